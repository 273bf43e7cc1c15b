// gsys_internal.h -- private glue between the host service (gsys_host.cpp) and the workload
// launchers (gsys_kernels.cu) built into the same libgsys.so.  Not part of the C-ABI.
#pragma once
#include <stddef.h>
#include <stdint.h>

struct gsys_dev_ctx;

// device pointer of the current device's instance context, or nullptr before gsys_init()
gsys_dev_ctx* gsys_internal_ctx_d();
int gsys_internal_nslots();

// pinned host ranges owned by the library (staging): the service resolves them without the driver
void gsys_internal_register_host_range(const void* p, size_t n, int add);

// gsys_launch for the library's own kernels: kernel_sites = false skips the reset of the
// kernel-scope call-site records (for kernels that make no kernel-granularity call)
int gsys_internal_launch(const void* kernel, uint32_t grid, uint32_t block, void** args, size_t smem, void* stream,
                         bool kernel_sites);
