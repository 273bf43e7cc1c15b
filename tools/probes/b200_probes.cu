// b200_probes.cu -- measurement probes for DESIGN.md / profiles (not part of the product path).
//   table4   : B200 analogue of the paper's Table IV (PAPER.md:26 P26.0-1, values lost in the
//              transcription): latency of one dependent cmp-swap / swap / atomic-add / acquire
//              load / relaxed load / plain load by one GPU thread, on device memory (HBM / L2) and
//              on pinned host-mapped memory (PCIe), at gpu and sys scope.
//   alu      : INT32 ALU peak (IADD3 / LOP3 / IMAD streams, independent chains, full occupancy).
//   smem     : shared-memory pipe peaks: conflict-free LDS.32 (wavefronts/s) and random LDS.U16
//              gathers over a 128 KB table (the DFA scan's access pattern).
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o /tmp/b200_probes b200_probes.cu
// Run:   /tmp/b200_probes            (one JSON line per measurement)
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e_)); exit(1); } } while (0)

__device__ __forceinline__ unsigned long long gtime() {
    unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t;
}

enum Op { LD_PLAIN = 0, LD_RELAXED_SYS, LD_ACQUIRE_SYS, LD_ACQUIRE_GPU, CAS_SYS, CAS_GPU, EXCH_SYS, EXCH_GPU,
          ADD_SYS, ADD_GPU, NOPS };
static const char* kOpName[NOPS] = {"load (plain, volatile)", "ld.relaxed.sys", "ld.acquire.sys", "ld.acquire.gpu",
                                   "atom.cas.sys", "atom.cas.gpu", "atom.exch.sys", "atom.exch.gpu",
                                   "atom.add.sys", "atom.add.gpu"};

// one thread: n dependent operations on p[idx], idx derived from the previous result (value 0)
__global__ void chain_kernel(unsigned* p, int op, int n, unsigned long long* out) {
    unsigned v = 0;
    const unsigned long long t0 = gtime();
    for (int i = 0; i < n; i++) {
        unsigned* q = p + (v & 1u) * 16u;   // always p (v stays 0/1 -> even), but the address depends on v
        switch (op) {
            case LD_PLAIN: v = *(volatile unsigned*)q; break;
            case LD_RELAXED_SYS: asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(q) : "memory"); break;
            case LD_ACQUIRE_SYS: asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(q) : "memory"); break;
            case LD_ACQUIRE_GPU: asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(q) : "memory"); break;
            case CAS_SYS: asm volatile("atom.sys.global.cas.b32 %0, [%1], %2, %3;" : "=r"(v) : "l"(q), "r"(v), "r"(v) : "memory"); break;
            case CAS_GPU: asm volatile("atom.gpu.global.cas.b32 %0, [%1], %2, %3;" : "=r"(v) : "l"(q), "r"(v), "r"(v) : "memory"); break;
            case EXCH_SYS: asm volatile("atom.sys.global.exch.b32 %0, [%1], %2;" : "=r"(v) : "l"(q), "r"(v) : "memory"); break;
            case EXCH_GPU: asm volatile("atom.gpu.global.exch.b32 %0, [%1], %2;" : "=r"(v) : "l"(q), "r"(v) : "memory"); break;
            case ADD_SYS: asm volatile("atom.sys.global.add.u32 %0, [%1], 0;" : "=r"(v) : "l"(q) : "memory"); break;
            case ADD_GPU: asm volatile("atom.gpu.global.add.u32 %0, [%1], 0;" : "=r"(v) : "l"(q) : "memory"); break;
        }
        v &= 0u;
    }
    out[0] = gtime() - t0;
    out[1] = v;
}

template <int K>
__global__ void alu_kernel(unsigned* out, int iters, unsigned seed) {
    unsigned a[8];
#pragma unroll
    for (int j = 0; j < 8; j++) a[j] = seed ^ (threadIdx.x * 0x9e3779b9u + j);
    for (int i = 0; i < iters; i++) {
#pragma unroll
        for (int u = 0; u < 16; u++) {
#pragma unroll
            for (int j = 0; j < 8; j++) {
                if (K == 0) a[j] = a[j] + a[(j + 1) & 7] + 0x1234567u;          // IADD3
                else if (K == 1) a[j] = (a[j] & a[(j + 3) & 7]) ^ (a[(j + 5) & 7] | 0x55u);   // LOP3
                else a[j] = a[j] * 0x9e3779b1u + a[(j + 2) & 7];               // IMAD
            }
        }
    }
    unsigned r = 0;
#pragma unroll
    for (int j = 0; j < 8; j++) r ^= a[j];
    if (r == 0x12345u) out[0] = r;
}

// conflict-free 32-bit loads: lane l reads word (l + 32 k) -> one wavefront per warp instruction
__global__ void lds32_kernel(unsigned* out, int iters) {
    extern __shared__ unsigned sm[];
    for (int i = threadIdx.x; i < 8192; i += blockDim.x) sm[i] = i * 2654435761u;
    __syncthreads();
    unsigned acc = 0, idx = threadIdx.x & 31u;
    for (int i = 0; i < iters; i++) {
#pragma unroll
        for (int u = 0; u < 16; u++) {
            acc += sm[(idx + 32u * ((u + i) & 255u)) & 8191u];
        }
    }
    if (acc == 0x777u) out[0] = acc;
}

// random 16-bit gathers over a 128 KB table (the DFA scan's lookup pattern); each lane's address
// depends on its previous load, like a DFA chain; 16 independent chains per thread
__global__ void lds16_random_kernel(unsigned* out, int iters, unsigned nwords, unsigned sentinel) {
    extern __shared__ unsigned short t16[];
    for (unsigned i = threadIdx.x; i < nwords; i += blockDim.x) t16[i] = (unsigned short)((i * 2654435761u) >> 7);
    __syncthreads();
    const unsigned mask = nwords - 1u;   // power of two
    unsigned e[8];
#pragma unroll
    for (int j = 0; j < 8; j++) e[j] = (threadIdx.x * 7919u + j * 104729u) & mask;
    for (int i = 0; i < iters; i++) {
#pragma unroll
        for (int u = 0; u < 8; u++) {
#pragma unroll
            for (int j = 0; j < 8; j++) e[j] = (t16[e[j]] + u + j) & mask;
        }
    }
    unsigned r = 0;
#pragma unroll
    for (int j = 0; j < 8; j++) r ^= e[j];
    if (r == sentinel) out[0] = r;   // a run-time value: the chains cannot be optimised away
}

static float time_kernel(void (*launch)(void*), void* arg) {
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    launch(arg);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(a));
    launch(arg);
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, a, b));
    return ms;
}

struct AluArg { int k, blocks, threads, iters; unsigned* out; };
static void launch_alu(void* p) {
    AluArg* a = (AluArg*)p;
    if (a->k == 0) alu_kernel<0><<<a->blocks, a->threads>>>(a->out, a->iters, 1u);
    else if (a->k == 1) alu_kernel<1><<<a->blocks, a->threads>>>(a->out, a->iters, 1u);
    else alu_kernel<2><<<a->blocks, a->threads>>>(a->out, a->iters, 1u);
}
struct SmArg { int k, blocks, threads, iters; unsigned* out; unsigned nwords; };
static void launch_sm(void* p) {
    SmArg* a = (SmArg*)p;
    if (a->k == 0) lds32_kernel<<<a->blocks, a->threads, 8192 * 4>>>(a->out, a->iters);
    else lds16_random_kernel<<<a->blocks, a->threads, a->nwords * 2>>>(a->out, a->iters, a->nwords, 0x7fffffffu);
}

int main() {
    int sms = 0, clk = 0;
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
    CK(cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0));
    unsigned* dmem;
    unsigned* hmem;
    unsigned* hdev;
    unsigned long long* out;
    CK(cudaMalloc(&dmem, 4096));
    CK(cudaMemset(dmem, 0, 4096));
    CK(cudaHostAlloc(&hmem, 4096, cudaHostAllocMapped));
    for (int i = 0; i < 1024; i++) hmem[i] = 0;
    CK(cudaHostGetDevicePointer((void**)&hdev, hmem, 0));
    CK(cudaMallocManaged(&out, 64));
    // ---- table 4
    for (int m = 0; m < 2; m++) {
        unsigned* p = m == 0 ? dmem : hdev;
        for (int op = 0; op < NOPS; op++) {
            const int n = m == 0 ? 20000 : 2000;
            chain_kernel<<<1, 1>>>(p, op, 200, out);
            CK(cudaDeviceSynchronize());
            double best = 1e30;
            for (int r = 0; r < 5; r++) {
                chain_kernel<<<1, 1>>>(p, op, n, out);
                CK(cudaDeviceSynchronize());
                const double ns = (double)out[0] / n;
                if (ns < best) best = ns;
            }
            printf("{\"probe\": \"table4\", \"memory\": \"%s\", \"op\": \"%s\", \"ns_per_op\": %.1f, \"chain\": %d}\n",
                   m == 0 ? "device (HBM, L2-resident)" : "pinned host-mapped (PCIe)", kOpName[op], best, n);
            fflush(stdout);
        }
    }
    // ---- INT32 ALU peak
    const char* kn[3] = {"IADD3", "LOP3", "IMAD"};
    for (int k = 0; k < 3; k++) {
        AluArg a{k, sms * 2, 1024, 2000, (unsigned*)out};
        const float ms = time_kernel(launch_alu, &a);
        const double ops = (double)a.blocks * a.threads * a.iters * 16 * 8;
        printf("{\"probe\": \"alu\", \"op\": \"%s\", \"Tops_per_s\": %.2f, \"per_sm_per_clk\": %.1f, \"sm_clock_mhz_attr\": %d}\n",
               kn[k], ops / (ms * 1e-3) / 1e12, ops / (ms * 1e-3) / sms / (clk * 1e3), clk / 1000);
        fflush(stdout);
    }
    // ---- shared-memory pipe
    {
        SmArg a{0, sms * 2, 1024, 4000, (unsigned*)out, 0};
        const float ms = time_kernel(launch_sm, &a);
        const double warp_instr = (double)a.blocks * (a.threads / 32) * a.iters * 16;
        printf("{\"probe\": \"smem\", \"op\": \"LDS.32 conflict-free\", \"wavefronts_per_s\": %.3e, \"per_sm_per_clk\": %.2f, \"GBps\": %.0f}\n",
               warp_instr / (ms * 1e-3), warp_instr / (ms * 1e-3) / sms / (clk * 1e3), warp_instr * 128 / (ms * 1e-3) / 1e9);
        fflush(stdout);
    }
    {
        const unsigned nwords = 65536;       // 128 KB: about the scan's 116 KB wide DFA table
        CK(cudaFuncSetAttribute(lds16_random_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(nwords * 2)));
        SmArg a{1, sms, 512, 400, (unsigned*)out, nwords};
        const float ms = time_kernel(launch_sm, &a);
        const double lookups = (double)a.blocks * a.threads * a.iters * 8 * 8;
        printf("{\"probe\": \"smem\", \"op\": \"LDS.U16 random gather (128 KB table)\", \"lookups_per_s\": %.3e, \"per_sm_per_clk\": %.2f, \"warp_instr_per_sm_per_clk\": %.3f}\n",
               lookups / (ms * 1e-3), lookups / (ms * 1e-3) / sms / (clk * 1e3), lookups / 32 / (ms * 1e-3) / sms / (clk * 1e3));
        fflush(stdout);
    }
    return 0;
}
