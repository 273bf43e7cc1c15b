// hostlink_probe.cu -- how fast can SMs pull pinned host-mapped memory over PCIe on B200?
// Variants: per-thread cp.async 16 B (the wc_kernel's current staging), LDG.128, TMA bulk
// copies (cp.async.bulk ... mbarrier::complete_tx) of B bytes with S stages per CTA, and the copy
// engine (cudaMemcpyAsync).  Prints one JSON line per variant.
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <stdint.h>
#include <string.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); exit(1); } } while (0)

__device__ unsigned long long g_sink;

__global__ void k_ldg(const uint4* __restrict__ p, size_t n16, int unroll) {
    unsigned acc = 0;
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (; i + 3 * stride < n16; i += 4 * stride) {
        uint4 a = p[i], b = p[i + stride], c = p[i + 2 * stride], d = p[i + 3 * stride];
        acc += a.x ^ b.y ^ c.z ^ d.w;
    }
    for (; i < n16; i += stride) acc += p[i].x;
    if (acc == 0x12345678u) g_sink = acc;
}

// per-warp 2 KiB tiles by cp.async 16 B, double-buffered (the wc_kernel staging pattern)
__global__ void k_cpasync(const unsigned char* __restrict__ p, size_t n, size_t per_block) {
    extern __shared__ __align__(16) unsigned char sm[];
    const unsigned lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nw = blockDim.x >> 5;
    unsigned char* st = sm + warp * 4096;
    const unsigned sbase = (unsigned)__cvta_generic_to_shared(st);
    const size_t b0 = (size_t)blockIdx.x * per_block, b1 = b0 + per_block < n ? b0 + per_block : n;
    unsigned acc = 0;
    size_t base = b0 + 2048 * warp;
    auto issue = [&](size_t at, unsigned buf) {
        for (int k = 0; k < 4; k++)
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(sbase + buf * 2048 + 512 * k + 16 * lane),
                         "l"(p + at + 512 * k + 16 * lane) : "memory");
    };
    if (base < b1) issue(base, 0);
    asm volatile("cp.async.commit_group;" ::: "memory");
    for (unsigned it = 0; base < b1; base += 2048 * nw, it ^= 1) {
        if (base + 2048 * nw < b1) issue(base + 2048 * nw, it ^ 1);
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 1;" ::: "memory");
        __syncwarp();
        acc += *(const unsigned*)(st + it * 2048 + lane * 64);
        __syncwarp();
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    if (acc == 0x12345678u) g_sink = acc;
}

// TMA bulk copies: one elected thread keeps S copies of B bytes in flight per CTA.
__global__ void k_bulk(const unsigned char* __restrict__ p, size_t n, size_t per_block, unsigned B, unsigned S) {
    extern __shared__ __align__(128) unsigned char sm[];
    __shared__ __align__(8) unsigned long long mbar[16];
    const size_t b0 = (size_t)blockIdx.x * per_block, b1 = b0 + per_block < n ? b0 + per_block : n;
    const unsigned nchunks = (unsigned)((b1 > b0 ? b1 - b0 : 0) / B);
    if (threadIdx.x == 0) {
        for (unsigned s = 0; s < S; s++)
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"((unsigned)__cvta_generic_to_shared(&mbar[s])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    unsigned acc = 0;
    auto issue = [&](unsigned c) {
        const unsigned s = c % S;
        const unsigned mb = (unsigned)__cvta_generic_to_shared(&mbar[s]);
        const unsigned dst = (unsigned)__cvta_generic_to_shared(sm + (size_t)s * B);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(mb), "r"(B) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     :: "r"(dst), "l"(p + b0 + (size_t)c * B), "r"(B), "r"(mb) : "memory");
    };
    if (threadIdx.x == 0)
        for (unsigned c = 0; c < S && c < nchunks; c++) issue(c);
    for (unsigned c = 0; c < nchunks; c++) {
        const unsigned s = c % S, ph = (c / S) & 1u;
        const unsigned mb = (unsigned)__cvta_generic_to_shared(&mbar[s]);
        asm volatile("{ .reg .pred P; WAIT_%=: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1; @!P bra WAIT_%=; }"
                     :: "r"(mb), "r"(ph) : "memory");
        acc += *(const unsigned*)(sm + (size_t)s * B + 4 * (threadIdx.x % (B / 4)));
        __syncthreads();   // everyone is done with stage s
        if (threadIdx.x == 0 && c + S < nchunks) issue(c + S);
    }
    if (acc == 0x12345678u) g_sink = acc;
}

static float timeit(cudaEvent_t a, cudaEvent_t b) { float ms; CK(cudaEventElapsedTime(&ms, a, b)); return ms; }

int main(int argc, char** argv) {
    const size_t n = (size_t)1 << 30;
    unsigned char* h;
    CK(cudaHostAlloc((void**)&h, n, cudaHostAllocMapped | cudaHostAllocPortable));
    for (size_t i = 0; i < n; i += 4096) memset(h + i, (int)(i >> 12), 4096);
    unsigned char* hd;
    CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
    unsigned char* d;
    CK(cudaMalloc((void**)&d, n));
    int sms;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    const int reps = 3;
    // copy engine
    CK(cudaMemcpy(d, h, n, cudaMemcpyHostToDevice));
    CK(cudaEventRecord(e0));
    for (int r = 0; r < reps; r++) CK(cudaMemcpyAsync(d, h, n, cudaMemcpyHostToDevice));
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    printf("{\"variant\": \"copy_engine\", \"GBps\": %.2f}\n", reps * n / (timeit(e0, e1) / 1e3) / 1e9);
    const bool only_mix = argc > 1;
    for (int bps : {1, 2, 4}) for (int th : {256, 512, 1024}) {
        if (only_mix) break;
        const int blocks = sms * bps;
        k_ldg<<<blocks, th>>>((const uint4*)hd, n / 16, 4);
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e0));
        for (int r = 0; r < reps; r++) k_ldg<<<blocks, th>>>((const uint4*)hd, n / 16, 4);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        printf("{\"variant\": \"ldg128\", \"blocks\": %d, \"threads\": %d, \"GBps\": %.2f}\n", blocks, th,
               reps * n / (timeit(e0, e1) / 1e3) / 1e9);
    }
    for (int bps : {1, 2, 4}) for (int th : {256, 512}) {
        if (only_mix) break;
        const int blocks = sms * bps;
        const size_t smem = (size_t)(th / 32) * 4096;
        CK(cudaFuncSetAttribute(k_cpasync, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        size_t per = (n / blocks + 2047) / 2048 * 2048;
        k_cpasync<<<blocks, th, smem>>>(hd, n, per);
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e0));
        for (int r = 0; r < reps; r++) k_cpasync<<<blocks, th, smem>>>(hd, n, per);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        printf("{\"variant\": \"cp_async16\", \"blocks\": %d, \"threads\": %d, \"GBps\": %.2f}\n", blocks, th,
               reps * n / (timeit(e0, e1) / 1e3) / 1e9);
    }
    for (unsigned B : {4096u, 16384u, 32768u}) for (unsigned S : {2u, 4u, 8u}) for (int bps : {1, 2}) {
        if (only_mix) break;
        const size_t smem = (size_t)B * S;
        if (smem * bps > 200 * 1024) continue;
        const int blocks = sms * bps;
        CK(cudaFuncSetAttribute(k_bulk, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        size_t per = (n / blocks + B - 1) / B * B;
        k_bulk<<<blocks, 128, smem>>>(hd, n, per, B, S);
        CK(cudaGetLastError());
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e0));
        for (int r = 0; r < reps; r++) k_bulk<<<blocks, 128, smem>>>(hd, n, per, B, S);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        printf("{\"variant\": \"tma_bulk\", \"bytes\": %u, \"stages\": %u, \"blocks\": %d, \"GBps\": %.2f}\n", B, S, blocks,
               reps * n / (timeit(e0, e1) / 1e3) / 1e9);
    }
    // concurrency: SM reads (ldg128 over the first half) while the copy engine moves the second half
    if (argc > 1) {
        cudaStream_t s1, s2;
        CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
        CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
        for (double frac_ce : {0.0, 0.1, 0.2, 0.3, 0.5}) {
            const size_t nce = ((size_t)(n * frac_ce) / 4096) * 4096, nsm = n - nce;
            cudaEvent_t a0, a1, b1;
            CK(cudaEventCreate(&a0)); CK(cudaEventCreate(&a1)); CK(cudaEventCreate(&b1));
            CK(cudaDeviceSynchronize());
            CK(cudaEventRecord(a0, s1));
            CK(cudaStreamWaitEvent(s2, a0, 0));
            for (int r = 0; r < reps; r++) {
                if (nsm) k_ldg<<<sms * 2, 512, 0, s1>>>((const uint4*)hd, nsm / 16, 4);
                if (nce) CK(cudaMemcpyAsync(d + nsm, h + nsm, nce, cudaMemcpyHostToDevice, s2));
            }
            CK(cudaEventRecord(a1, s1));
            CK(cudaEventRecord(b1, s2));
            CK(cudaEventSynchronize(a1));
            CK(cudaEventSynchronize(b1));
            const float t1 = timeit(a0, a1), t2 = timeit(a0, b1);
            const float t = t1 > t2 ? t1 : t2;
            printf("{\"variant\": \"sm+ce\", \"ce_fraction\": %.2f, \"sm_ms\": %.3f, \"ce_ms\": %.3f, \"GBps\": %.2f}\n",
                   frac_ce, t1 / reps, t2 / reps, reps * n / (t / 1e3) / 1e9);
        }
    }
    fflush(stdout);
    return 0;
}
