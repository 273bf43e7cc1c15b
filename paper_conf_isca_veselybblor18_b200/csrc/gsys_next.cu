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

#include <vector>

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

// ------------------------------------------------------------------ config 4: memcached-style UDP GETs
// Layout (device): McEntry[nbuckets][bucket_cap] (keys zero-padded to 32 B), bucket fill counts,
// and a value heap.  One work-group per in-flight request: recvfrom -> parse -> FNV-1a bucket ->
// all threads compare the bucket's entries (up to 1024, the paper's large-bucket case, P32.33) ->
// reply assembled in the work-group's host-mapped buffer -> sendto (both WG, blocking, weak --
// the paper's choice, P32.29-30).
struct McEntry {
    uint4 k0, k1;
    unsigned klen, vlen;
    unsigned long long voff;
};
static_assert(sizeof(McEntry) == 48, "McEntry layout");

constexpr unsigned MC_IO_BYTES = 8192;       // per work-group: rx | tx | from | fromlen
constexpr unsigned MC_RX = 0, MC_TX = 2048, MC_FROM = 7168, MC_FROMLEN = 7296;
constexpr unsigned MC_MAXKEY = 32, MC_MAXVAL = 4096;

__host__ __device__ __forceinline__ unsigned mc_hash(const unsigned char* k, unsigned n) {
    unsigned h = 2166136261u;
    for (unsigned i = 0; i < n; i++) { h ^= k[i]; h *= 16777619u; }
    return h;
}

struct McArgs {
    const gsys_dev_ctx* ctx;
    const McEntry* entries;
    const unsigned* bucket_n;
    const unsigned char* heap;
    unsigned char* io;              // host-mapped [nwg][MC_IO_BYTES]
    const volatile unsigned* stop;  // host-mapped stop flag
    unsigned long long* stats;      // device [4]: served, misses, malformed, recv timeouts
    unsigned nbuckets, cap, gflags, send_gflags;
    int fd, pad_;
};

__device__ __forceinline__ unsigned be16(const unsigned char* p) { return ((unsigned)p[0] << 8) | p[1]; }
__device__ __forceinline__ void put_be16(unsigned char* p, unsigned v) { p[0] = (unsigned char)(v >> 8); p[1] = (unsigned char)v; }
__device__ __forceinline__ void put_be32(unsigned char* p, unsigned v) {
    p[0] = (unsigned char)(v >> 24); p[1] = (unsigned char)(v >> 16); p[2] = (unsigned char)(v >> 8); p[3] = (unsigned char)v;
}

__global__ void __launch_bounds__(256) mc_kernel(McArgs a) {
    __shared__ unsigned s_found, s_len, s_keylen, s_bucket, s_ok, s_done, s_fromlen;
    __shared__ __align__(16) unsigned char s_rx[80];      // frame + header + extras + key (<= 32 + 16 + 32)
    __shared__ __align__(16) unsigned char s_key[MC_MAXKEY];
    __shared__ gsys_token s_stok;   // the previous (non-blocking) reply's sendto
    if (threadIdx.x == 0) { s_stok.slot = 0u; s_stok.seq = 0u; }
    unsigned char* io = a.io + (size_t)blockIdx.x * MC_IO_BYTES;
    unsigned char* rx = io + MC_RX;
    unsigned char* tx = io + MC_TX;
    void* from = io + MC_FROM;
    unsigned* fromlen = reinterpret_cast<unsigned*>(io + MC_FROMLEN);
    const unsigned gf = a.gflags | GSYS_HOSTBUF;
    for (;;) {
        // the reply buffer and `from` may still be read by the previous non-blocking sendto: wait
        // for that request by its token, whatever slot this work-group's next call lands in
        if (a.send_gflags & GSYS_NONBLOCKING) gsys_wait_token(a.ctx, &s_stok, GSYS_WG);
        if (threadIdx.x == 0) *(volatile unsigned*)fromlen = 128u;
        const long long r = gsys_recvfrom(a.ctx, a.fd, rx, 2048, 0, from, fromlen, gf);   // producer: Bar2
        if (r < 0) {
            if (threadIdx.x == 0) {
                s_done = *a.stop;
                if (r == -EAGAIN || r == -EWOULDBLOCK) atomicAdd(&a.stats[3], 1ull);
            }
            __syncthreads();
            if (s_done) break;
            continue;
        }
        // the first 80 bytes of the datagram in one coalesced PCIe read (5 lanes x 16 B), then
        // parse from shared memory -- byte-wise volatile reads would cost one round trip each
        if (threadIdx.x < 5) reinterpret_cast<uint4*>(s_rx)[threadIdx.x] = reinterpret_cast<const uint4*>(rx)[threadIdx.x];
        if (threadIdx.x == 5) s_fromlen = *fromlen;
        __syncthreads();
        if (threadIdx.x == 0) {
            const unsigned char* v = s_rx;
            unsigned ok = r >= 32 && v[8] == 0x80 && v[9] == 0x00;
            const unsigned klen = be16(v + 10), ext = v[12];
            ok = ok && klen >= 1 && klen <= MC_MAXKEY && ext <= 16 && (long long)(32 + ext + klen) <= r;
            s_keylen = ok ? klen : 0u;
            for (unsigned i = 0; i < MC_MAXKEY; i++) s_key[i] = (ok && i < klen) ? v[32 + ext + i] : 0u;
            s_bucket = ok ? mc_hash(s_key, klen) % a.nbuckets : 0u;
            s_ok = ok;
            s_found = 0xffffffffu;
            if (!ok) atomicAdd(&a.stats[2], 1ull);
        }
        __syncthreads();
        if (!s_ok) continue;
        // parallel bucket scan
        const uint4 K0 = *reinterpret_cast<const uint4*>(s_key), K1 = *reinterpret_cast<const uint4*>(s_key + 16);
        const unsigned n = a.bucket_n[s_bucket];
        const McEntry* B = a.entries + (size_t)s_bucket * a.cap;
        for (unsigned i = threadIdx.x; i < n; i += blockDim.x) {
            const McEntry e = B[i];
            if (e.klen == s_keylen && e.k0.x == K0.x && e.k0.y == K0.y && e.k0.z == K0.z && e.k0.w == K0.w &&
                e.k1.x == K1.x && e.k1.y == K1.y && e.k1.z == K1.z && e.k1.w == K1.w)
                atomicMin(&s_found, i);
        }
        __syncthreads();
        const bool hit = s_found != 0xffffffffu;
        const McEntry* e = hit ? B + s_found : nullptr;
        const unsigned vlen = hit ? e->vlen : 0u;

        // reply: UDP frame header + binary response header (+ flags + value | "Not found")
        if (threadIdx.x == 0) {
            const unsigned char* v = s_rx;
            __align__(16) unsigned char h[48];
            for (int i = 0; i < 48; i++) h[i] = 0;
            h[0] = v[0]; h[1] = v[1];                 // request id
            put_be16(h + 4, 1u);                      // total datagrams
            h[8] = 0x81;                              // magic: response
            h[9] = 0x00;                              // opcode: GET
            h[12] = hit ? 4 : 0;                      // extras length (flags)
            put_be16(h + 14, hit ? 0u : 1u);          // status: 0 ok, 1 key not found
            put_be32(h + 16, hit ? 4u + vlen : 9u);   // total body
            for (int i = 0; i < 4; i++) h[20 + i] = v[20 + i];   // opaque
            if (!hit) {
                const char nf[9] = {'N', 'o', 't', ' ', 'f', 'o', 'u', 'n', 'd'};
                for (int i = 0; i < 9; i++) h[32 + i] = (unsigned char)nf[i];
            }
            for (int i = 0; i < 2; i++) reinterpret_cast<uint4*>(tx)[i] = reinterpret_cast<const uint4*>(h)[i];
            if (!hit) reinterpret_cast<uint4*>(tx)[2] = reinterpret_cast<const uint4*>(h)[2];
            else *reinterpret_cast<unsigned*>(tx + 32) = 0u;     // flags
            s_len = hit ? 36u + vlen : 41u;
            atomicAdd(&a.stats[0], 1ull);
            if (!hit) atomicAdd(&a.stats[1], 1ull);
        }
        if (hit) {
            const unsigned char* src = a.heap + e->voff;
            for (unsigned i = threadIdx.x; i < vlen; i += blockDim.x) tx[36 + i] = src[i];
        }
        // consumer call: Bar1 (the reply is complete) is kept under relaxed ordering
        gsys_sendto(a.ctx, a.fd, tx, s_len, 0, from, s_fromlen, a.send_gflags | GSYS_HOSTBUF, &s_stok);
        __syncthreads();
    }
}

// ------------------------------------------------------------------ row f3: Fig. 8 permutation + pwrite
// PAPER.md:26 sec. VII "Blocking and ordering strategies": work-groups of 1024 work-items
// independently permute 8 KB blocks (a DES-like permutation step, repeated `iters` times) and
// write each result to a file with a work-group pwrite; blocking x ordering is the study.
struct PermArgs {
    const gsys_dev_ctx* ctx;
    const unsigned char* in;          // DEVICE [nblocks][bs]
    const unsigned short* perm;       // DEVICE [bs] permutation: out[i] = in[perm[i]]
    unsigned char* staging;           // host-mapped [nblocks][bs] (one line per block: no reuse hazard)
    unsigned long long file_off;
    unsigned nblocks, bs, iters, gflags;
    int fd, pad_;
};

__global__ void __launch_bounds__(1024) perm_kernel(PermArgs a) {
    extern __shared__ __align__(16) unsigned char psm[];   // [bs] x 2 + perm [bs] u16
    unsigned char* b0 = psm;
    unsigned char* b1 = psm + a.bs;
    unsigned short* pm = reinterpret_cast<unsigned short*>(psm + 2 * a.bs);
    for (unsigned i = threadIdx.x; i < a.bs; i += blockDim.x) pm[i] = a.perm[i];
    for (unsigned blk = blockIdx.x; blk < a.nblocks; blk += gridDim.x) {
        const unsigned char* src = a.in + (size_t)blk * a.bs;
        for (unsigned i = threadIdx.x; i < a.bs / 16u; i += blockDim.x)
            reinterpret_cast<uint4*>(b0)[i] = reinterpret_cast<const uint4*>(src)[i];
        __syncthreads();
        unsigned char* cur = b0;
        unsigned char* nxt = b1;
        for (unsigned it = 0; it < a.iters; it++) {
            for (unsigned i = threadIdx.x; i < a.bs; i += blockDim.x) nxt[i] = cur[pm[i]];
            __syncthreads();
            unsigned char* t = cur; cur = nxt; nxt = t;
        }
        unsigned char* out = a.staging + (size_t)blk * a.bs;
        for (unsigned i = threadIdx.x; i < a.bs / 16u; i += blockDim.x)
            reinterpret_cast<uint4*>(out)[i] = reinterpret_cast<const uint4*>(cur)[i];
        // consumer call: Bar1 always (the block is complete); Bar2 only when strong
        gsys_pwrite(a.ctx, a.fd, out, a.bs, (long long)(a.file_off + (unsigned long long)blk * a.bs),
                    a.gflags | GSYS_HOSTBUF);
        __syncthreads();   // both shared buffers are reused by the next block
    }
}

// ------------------------------------------------------------------ row f4: Fig. 9 polling contention
// PAPER.md:28 sec. VII "Polling/halt-resume and memory contention": GPU threads poll `nlines`
// distinct 64 B lines (as completion polls would) for `ns` nanoseconds while the host measures its
// own memory throughput.  host = 1 polls pinned host-mapped lines (each poll is a PCIe read, the
// B200 analogue of spilling past the APU's L2); host = 0 polls device lines (L2-resident).
__global__ void poll_kernel(const unsigned long long* lines, unsigned nlines, unsigned long long ns,
                            unsigned long long* sink) {
    const unsigned tid = blockIdx.x * blockDim.x + threadIdx.x;
    const unsigned long long* p = lines + (size_t)(tid % nlines) * 8;
    const unsigned long long end = gsys::globaltimer() + ns;
    unsigned long long mx = 0, polls = 0;
    while (gsys::globaltimer() < end) {
        const unsigned long long v = gsys::ld_relaxed_sys(p);   // system scope: sees host stores
        mx = v > mx ? v : mx;
        polls++;
    }
    atomicAdd(sink, polls);
    atomicMax(sink + 1, mx);
}

}  // namespace

extern "C" {

int gsys_poll_storm(const void* lines, uint32_t nlines, uint32_t nthreads, uint64_t ns, uint64_t* d_sink,
                    void* stream) {
    if (!lines || !nlines || !nthreads || !d_sink) return -EINVAL;
    const unsigned bs = 256, nb = (nthreads + bs - 1) / bs;
    poll_kernel<<<nb, bs, 0, (cudaStream_t)stream>>>(reinterpret_cast<const unsigned long long*>(lines), nlines, ns,
                                                    reinterpret_cast<unsigned long long*>(d_sink));
    return cudaGetLastError() == cudaSuccess ? 0 : -EIO;
}


int gsys_perm_pwrite(const uint8_t* d_in, const uint16_t* d_perm, uint32_t nblocks, uint32_t block_bytes,
                     uint32_t iters, uint8_t* staging, int32_t fd, uint64_t file_off, uint32_t gflags, uint32_t grid,
                     void* stream) {
    gsys_dev_ctx* ctx = gsys_internal_ctx_d();
    if (!ctx) return -ENODEV;
    if (!d_in || !d_perm || !staging || !nblocks || !block_bytes || block_bytes % 16 || block_bytes > 16384)
        return -EINVAL;
    if ((gflags & GSYS_GRAN_MASK) != GSYS_WG) return -EINVAL;
    PermArgs a;
    memset(&a, 0, sizeof a);
    a.ctx = ctx;
    a.in = d_in;
    a.perm = d_perm;
    a.staging = staging;
    a.file_off = file_off;
    a.nblocks = nblocks;
    a.bs = block_bytes;
    a.iters = iters;
    a.gflags = gflags;
    a.fd = fd;
    const size_t smem = 4ull * block_bytes;
    if (smem > 48 * 1024 &&
        cudaFuncSetAttribute((const void*)perm_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
            cudaSuccess)
        return -EINVAL;
    if (grid == 0 || grid > nblocks) grid = nblocks;
    void* args[] = {&a};
    return gsys_launch((const void*)perm_kernel, grid, 1, 1, 1024, 1, 1, args, smem, stream);
}


int gsys_mc_build(const uint8_t* keys, const uint32_t* key_off, const uint8_t* key_len, const uint8_t* vals,
                  const uint64_t* val_off, const uint32_t* val_len, uint32_t n, uint32_t nbuckets, uint32_t bucket_cap,
                  void* d_entries, uint32_t* d_bucket_n, uint8_t* d_heap, uint64_t heap_bytes) {
    if (!n || !nbuckets || !bucket_cap || !keys || !key_off || !key_len || !vals || !val_off || !val_len ||
        !d_entries || !d_bucket_n || !d_heap)
        return -EINVAL;
    std::vector<McEntry> ent((size_t)nbuckets * bucket_cap);
    memset(ent.data(), 0, ent.size() * sizeof(McEntry));
    std::vector<uint32_t> cnt(nbuckets, 0);
    uint64_t hend = 0;
    for (uint32_t i = 0; i < n; i++) {
        const unsigned kl = key_len[i];
        if (kl < 1 || kl > MC_MAXKEY || val_len[i] > MC_MAXVAL) return -EINVAL;
        const unsigned b = mc_hash(keys + key_off[i], kl) % nbuckets;
        if (cnt[b] >= bucket_cap) return -E2BIG;
        McEntry& e = ent[(size_t)b * bucket_cap + cnt[b]++];
        unsigned char kb[32] = {0};
        memcpy(kb, keys + key_off[i], kl);
        memcpy(&e.k0, kb, 16);
        memcpy(&e.k1, kb + 16, 16);
        e.klen = kl;
        e.vlen = val_len[i];
        e.voff = val_off[i];
        if (val_off[i] + val_len[i] > hend) hend = val_off[i] + val_len[i];
    }
    if (hend > heap_bytes) return -EINVAL;
    if (cudaMemcpy(d_entries, ent.data(), ent.size() * sizeof(McEntry), cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(d_bucket_n, cnt.data(), nbuckets * 4, cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(d_heap, vals, hend, cudaMemcpyHostToDevice) != cudaSuccess)
        return -EIO;
    return 0;
}

uint64_t gsys_mc_entries_bytes(uint32_t nbuckets, uint32_t bucket_cap) {
    return (uint64_t)nbuckets * bucket_cap * sizeof(McEntry);
}

int gsys_mc_serve(int32_t fd, const void* d_entries, const uint32_t* d_bucket_n, const uint8_t* d_heap,
                  uint32_t nbuckets, uint32_t bucket_cap, uint32_t nwg, uint8_t* io, const uint32_t* stop,
                  uint64_t* d_stats, uint32_t gflags, uint32_t send_gflags, void* stream) {
    gsys_dev_ctx* ctx = gsys_internal_ctx_d();
    if (!ctx) return -ENODEV;
    if (!d_entries || !d_bucket_n || !d_heap || !nbuckets || !bucket_cap || !nwg || !io || !stop || !d_stats)
        return -EINVAL;
    if ((gflags & GSYS_GRAN_MASK) != GSYS_WG || (gflags & GSYS_NONBLOCKING)) return -EINVAL;
    if ((send_gflags & GSYS_GRAN_MASK) != GSYS_WG) return -EINVAL;
    McArgs a;
    memset(&a, 0, sizeof a);
    a.ctx = ctx;
    a.entries = reinterpret_cast<const McEntry*>(d_entries);
    a.bucket_n = d_bucket_n;
    a.heap = d_heap;
    a.io = io;
    a.stop = stop;
    a.stats = reinterpret_cast<unsigned long long*>(d_stats);
    a.nbuckets = nbuckets;
    a.cap = bucket_cap;
    a.gflags = gflags;
    a.send_gflags = send_gflags;
    a.fd = fd;
    void* args[] = {&a};
    return gsys_launch((const void*)mc_kernel, nwg, 1, 1, 256, 1, 1, args, 0, stream);
}



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
