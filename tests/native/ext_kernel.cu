// A kernel compiled OUTSIDE libgsys (its own module and CUDA runtime), using only the public
// device API (include/gsys_device.cuh), launched through gsys_launch_cu.  Test-only.
//
// Each block: lane 0 of warp w issues a work-item NON-BLOCKING pread of chunk (block, w) into
// dbuf and leaves its completion token in shared memory; consecutive calls therefore come from
// different warps (different hardware slots).  After a barrier, lane 0 of the NEXT warp waits on
// that token -- another thread's request -- and sums the chunk's bytes.  Then the whole block
// issues one blocking work-group pread and sums that buffer cooperatively.
#include <cuda_runtime.h>

#include "gsys_device.cuh"

struct ExtArgs {
    const gsys_dev_ctx* ctx;
    unsigned char* dbuf;        // [blocks * (nwarps + 1) * len]
    long long* ret;             // [blocks * (nwarps + 1)]: token result (WI) / pread return (WG)
    unsigned long long* sum;    // [blocks * (nwarps + 1)]: byte sums
    unsigned long long size;
    unsigned len;
    int fd;
};

__global__ void ext_nb_relay(ExtArgs a) {
    __shared__ gsys_token s_tok[32];
    __shared__ unsigned long long s_sum;
    const unsigned warp = threadIdx.x / 32, lane = threadIdx.x % 32, nw = blockDim.x / 32;
    const unsigned long long base = (unsigned long long)blockIdx.x * (nw + 1);
    for (unsigned w = 0; w < nw; w++) {      // one call after the other, each from another warp
        if (warp == w && lane == 0) {
            const unsigned long long i = base + w;
            gsys_pread(a.ctx, a.fd, a.dbuf + i * a.len, a.len, (long long)((i * a.len) % a.size),
                       GSYS_WI | GSYS_NONBLOCKING, &s_tok[w]);
        }
        __syncthreads();
    }
    if (lane == 0) {
        const unsigned w = (warp + nw - 1) % nw;          // the previous warp's request
        const long long r = gsys_wait_token(a.ctx, &s_tok[w], GSYS_WI);
        const unsigned long long i = base + w;
        unsigned long long acc = 0;
        for (long long k = 0; k < (r > 0 ? r : 0); k++) acc += a.dbuf[i * a.len + k];
        a.ret[i] = r;
        a.sum[i] = acc;
    }
    const unsigned long long j = base + nw;
    const long long r = gsys_pread(a.ctx, a.fd, a.dbuf + j * a.len, a.len, (long long)((j * a.len) % a.size),
                                   GSYS_WG | GSYS_BLOCKING | GSYS_RELAXED);
    if (threadIdx.x == 0) s_sum = 0;
    __syncthreads();
    unsigned long long acc = 0;
    for (long long k = threadIdx.x; k < (r > 0 ? r : 0); k += blockDim.x) acc += a.dbuf[j * a.len + k];
    atomicAdd(&s_sum, acc);
    __syncthreads();
    if (threadIdx.x == 0) { a.ret[j] = r; a.sum[j] = s_sum; }
}

// Work-item blocking preads into device memory from a partial, diverged set of lanes (thread t
// calls unless t % 3 == 0) with per-lane lengths around the warp-copy limit (lengths from `lens`,
// indexed by lane), then one kernel-scope blocking pread of klen bytes into kbuf that every block
// sums after the call (the first-arriving block copied it before releasing the others).
struct MixArgs {
    const gsys_dev_ctx* ctx;
    unsigned char* dbuf;        // [threads_total * stride]
    long long* ret;             // [threads_total] (-2^40 if the thread did not call)
    unsigned long long* sum;    // [threads_total]
    const unsigned* lens;       // [32]
    unsigned char* kbuf;        // [klen]
    long long* kret;            // [blocks]
    unsigned long long* ksum;   // [blocks]
    unsigned long long size, stride, klen;
    int fd;
};

__global__ void ext_wi_mixed(MixArgs a) {
    const unsigned long long t = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x;
    const unsigned lane = threadIdx.x % 32;
    if (t % 3 != 0) {
        const unsigned len = a.lens[lane];
        const long long off = (long long)((t * 4099ull) % a.size);
        const long long r = gsys_pread(a.ctx, a.fd, a.dbuf + t * a.stride, len, off, GSYS_WI | GSYS_BLOCKING);
        unsigned long long acc = 0;
        for (long long k = 0; k < (r > 0 ? r : 0); k++) acc += a.dbuf[t * a.stride + k];
        a.ret[t] = r;
        a.sum[t] = acc;
    }
    __syncthreads();
    const long long r = gsys_pread(a.ctx, a.fd, a.kbuf, a.klen, 12345, GSYS_KERNEL | GSYS_BLOCKING | GSYS_RELAXED);
    __shared__ unsigned long long s_sum;
    if (threadIdx.x == 0) s_sum = 0;
    __syncthreads();
    unsigned long long acc = 0;
    for (long long k = threadIdx.x; k < (r > 0 ? r : 0); k += blockDim.x) acc += a.kbuf[k];
    atomicAdd(&s_sum, acc);
    __syncthreads();
    if (threadIdx.x == 0) { a.kret[blockIdx.x] = r; a.ksum[blockIdx.x] = s_sum; }
}

extern "C" int ext_function_mixed(void** f) {
    return cudaGetFuncBySymbol(reinterpret_cast<cudaFunction_t*>(f), reinterpret_cast<const void*>(ext_wi_mixed)) ==
                   cudaSuccess ? 0 : -1;
}

extern "C" int ext_function(void** f) {
    return cudaGetFuncBySymbol(reinterpret_cast<cudaFunction_t*>(f), reinterpret_cast<const void*>(ext_nb_relay)) ==
                   cudaSuccess ? 0 : -1;
}
