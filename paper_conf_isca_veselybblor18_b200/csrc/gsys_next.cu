// gsys_next.cu -- sm_100a kernels of the §8(f) "next" rows and their C-ABI launchers.
//
//   amr_kernel   memory management (config 5a, sec. VIII-A miniamr): each work-group
//                owns one block of an AMR-style mesh; per iteration it smooths its device field,
//                reads the process RSS with a GPU-issued pread of /proc/self/statm ("everything is
//                a file", P16.46; ru_maxrss is only the peak -- reading A12) plus getrusage, and
//                when its block is coarsened (refinement level 0) and RSS is above the watermark it
//                releases the block's host mirror with madvise(MADV_DONTNEED) at work-group
//                granularity, non-blocking, weak ordering (P28.29-36).
//   sig_kernel   signals (config 5b, sec. VIII-B signal-search): each work-group counts
//                the occurrences of a key in its data block, publishes the count, and notifies the
//                host with rt_sigqueueinfo(pid, sig, {SI_QUEUE, si_value = work-group id}) at
//                work-group granularity, non-blocking (P30.12-21); a host consumer sigwaits and
//                post-processes each block as soon as its signal arrives (the CPU phase overlaps
//                the GPU search).

#include <cuda_runtime.h>
#include <errno.h>
#include <stdint.h>
#include <string.h>
#include <sys/mman.h>

#include "gsys.h"
#include "gsys_device.cuh"
#include "gsys_internal.h"

namespace {

// ------------------------------------------------------------------ config 5a: AMR + madvise
struct AmrArgs {
    const gsys_dev_ctx* ctx;
    unsigned long long host_mesh;     // host address of the mesh (pageable; never dereferenced here)
    unsigned long long block_bytes;
    const unsigned char* levels;      // [iters][nblocks] refinement level, 0 = coarsened
    float* field;                     // [2][nblocks][fwords] device working field
    unsigned char* statm_buf;         // host-mapped [nblocks][128] pread target
    unsigned* released;               // [nblocks]: iteration+1 at which the block was released
    long long* rss;                   // [iters]: resident bytes seen by work-group 0
    long long* maxrss;                // [iters]: ru_maxrss (KiB) seen by work-group 0
    unsigned long long watermark;
    unsigned long long page_bytes;
    unsigned nblocks, iters, fwords, gflags;
    int statm_fd, pad_;
};

__device__ long long parse_statm_resident_pages(const unsigned char* b, long long n) {
    // "size resident shared ..." in pages: the second decimal field
    long long i = 0, field = 0, v = 0;
    bool in_num = false;
    for (; i < n; i++) {
        const unsigned c = b[i];
        if (c >= '0' && c <= '9') {
            if (!in_num) { in_num = true; v = 0; }
            v = v * 10 + (c - '0');
        } else if (in_num) {
            in_num = false;
            if (++field == 2) return v;
        }
    }
    return in_num && field == 1 ? v : -1;
}

__global__ void __launch_bounds__(256) amr_kernel(AmrArgs a) {
    const unsigned b = blockIdx.x;
    if (b >= a.nblocks) return;
    __shared__ long long s_rss;
    alignas(16) unsigned char ru[160];
    for (unsigned t = 0; t < a.iters; t++) {
        // stencil step on the device field of this block (the "compute" between system calls)
        const float* src = a.field + ((size_t)(t & 1) * a.nblocks + b) * a.fwords;
        float* dst = a.field + ((size_t)((t + 1) & 1) * a.nblocks + b) * a.fwords;
        for (unsigned i = threadIdx.x; i < a.fwords; i += blockDim.x) {
            const float l = src[i > 0 ? i - 1 : i], c = src[i], r = src[i + 1 < a.fwords ? i + 1 : i];
            dst[i] = 0.25f * l + 0.5f * c + 0.25f * r;
        }
        // resident set size through the file system: pread(/proc/self/statm) at WG granularity
        unsigned char* sb = a.statm_buf + (size_t)b * 128;
        const long long n = gsys_pread(a.ctx, a.statm_fd, sb, 127, 0, GSYS_WG | GSYS_BLOCKING | GSYS_RELAXED | GSYS_HOSTBUF);
        if (threadIdx.x == 0) {
            const long long pages = n > 0 ? parse_statm_resident_pages(sb, n) : -1;
            s_rss = pages >= 0 ? pages * (long long)a.page_bytes : -1;
        }
        const long long gr = gsys_getrusage(a.ctx, 0 /* RUSAGE_SELF */, ru, GSYS_WG | GSYS_BLOCKING | GSYS_RELAXED);
        __syncthreads();
        if (b == 0 && threadIdx.x == 0) {
            a.rss[t] = s_rss;
            a.maxrss[t] = gr == 0 ? *reinterpret_cast<const long long*>(ru + 32) : -1;   // ru_maxrss (KiB)
        }
        // release the host mirror of a coarsened block once RSS is above the watermark
        const bool release = a.levels[(size_t)t * a.nblocks + b] == 0 && a.released[b] == 0u &&
                             s_rss >= (long long)a.watermark;
        if (release) {   // uniform across the work-group
            gsys_madvise(a.ctx, (void*)(a.host_mesh + (unsigned long long)b * a.block_bytes), (size_t)a.block_bytes,
                         MADV_DONTNEED, a.gflags);
            if (threadIdx.x == 0) a.released[b] = t + 1u;
        }
        __syncthreads();
    }
}

// ------------------------------------------------------------------ config 5b: signal-search
struct SigArgs {
    const gsys_dev_ctx* ctx;
    const unsigned char* data;        // [nblocks][block_bytes]
    unsigned* counts;                 // [nblocks] (host-mapped or device)
    unsigned long long block_bytes;
    unsigned char key[16];
    unsigned keylen, nblocks, gflags;
    int tgid, sig, uid;
};

__global__ void __launch_bounds__(256) sig_kernel(SigArgs a) {
    const unsigned b = blockIdx.x;
    if (b >= a.nblocks) return;
    __shared__ unsigned s_count;
    if (threadIdx.x == 0) s_count = 0;
    __syncthreads();
    const unsigned char* d = a.data + (size_t)b * a.block_bytes;
    unsigned cnt = 0;
    const unsigned long long last = a.block_bytes >= a.keylen ? a.block_bytes - a.keylen : 0;
    for (unsigned long long i = threadIdx.x; i <= last && a.block_bytes >= a.keylen; i += blockDim.x) {
        bool m = true;
        for (unsigned k = 0; k < a.keylen && m; k++) m = d[i + k] == a.key[k];
        cnt += m ? 1u : 0u;
    }
    atomicAdd(&s_count, cnt);
    __syncthreads();
    if (threadIdx.x == 0) {
        *(volatile unsigned*)&a.counts[b] = s_count;
        __threadfence_system();
    }
    // siginfo for SI_QUEUE (x86-64 Linux layout): signo, errno, code, pad, pid, uid, sigval
    alignas(16) int si[32];
    for (int k = 0; k < 32; k++) si[k] = 0;
    si[0] = a.sig;
    si[2] = -1;            // SI_QUEUE
    si[4] = a.tgid;
    si[5] = a.uid;
    si[6] = (int)b;        // si_value.sival_int = work-group id
    gsys_rt_sigqueueinfo(a.ctx, a.tgid, a.sig, si, a.gflags);
}

}  // namespace

extern "C" {

int gsys_amr_release(uint64_t host_mesh, uint32_t nblocks, uint64_t block_bytes, const uint8_t* d_levels,
                     uint32_t iters, int32_t statm_fd, uint64_t watermark_bytes, uint64_t page_bytes, float* d_field,
                     uint32_t field_words, uint8_t* statm_buf, uint32_t* d_released, int64_t* d_rss, int64_t* d_maxrss,
                     uint32_t gflags, void* stream) {
    gsys_dev_ctx* ctx = gsys_internal_ctx_d();
    if (!ctx) return -ENODEV;
    if (!nblocks || !iters || !d_levels || !d_field || !statm_buf || !d_released || !d_rss || !d_maxrss)
        return -EINVAL;
    if ((gflags & GSYS_GRAN_MASK) != GSYS_WG) return -EINVAL;
    AmrArgs a;
    memset(&a, 0, sizeof a);
    a.ctx = ctx;
    a.host_mesh = host_mesh;
    a.block_bytes = block_bytes;
    a.levels = d_levels;
    a.field = d_field;
    a.statm_buf = statm_buf;
    a.released = d_released;
    a.rss = reinterpret_cast<long long*>(d_rss);
    a.maxrss = reinterpret_cast<long long*>(d_maxrss);
    a.watermark = watermark_bytes;
    a.page_bytes = page_bytes ? page_bytes : 4096;
    a.nblocks = nblocks;
    a.iters = iters;
    a.fwords = field_words;
    a.gflags = gflags;
    a.statm_fd = statm_fd;
    void* args[] = {&a};
    return gsys_launch((const void*)amr_kernel, nblocks, 1, 1, 256, 1, 1, args, 0, stream);
}

int gsys_signal_search(const uint8_t* d_data, uint32_t nblocks, uint64_t block_bytes, const uint8_t* key,
                       uint32_t keylen, int32_t tgid, int32_t sig, int32_t uid, uint32_t* counts, uint32_t gflags,
                       void* stream) {
    gsys_dev_ctx* ctx = gsys_internal_ctx_d();
    if (!ctx) return -ENODEV;
    if (!d_data || !nblocks || !key || keylen == 0 || keylen > 16 || !counts) return -EINVAL;
    if ((gflags & GSYS_GRAN_MASK) != GSYS_WG) return -EINVAL;
    SigArgs a;
    memset(&a, 0, sizeof a);
    a.ctx = ctx;
    a.data = d_data;
    a.counts = counts;
    a.block_bytes = block_bytes;
    memcpy(a.key, key, keylen);
    a.keylen = keylen;
    a.nblocks = nblocks;
    a.gflags = gflags;
    a.tgid = tgid;
    a.sig = sig;
    a.uid = uid;
    void* args[] = {&a};
    return gsys_launch((const void*)sig_kernel, nblocks, 1, 1, 256, 1, 1, args, 0, stream);
}

}  // extern "C"
