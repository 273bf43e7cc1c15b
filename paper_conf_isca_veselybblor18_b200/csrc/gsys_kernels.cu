// gsys_kernels.cu -- sm_100a kernels of the hot path and their C-ABI launchers.
//
//   wc_kernel     wordcount + grep -F -l over files read with work-group preads issued from the
//                 GPU (sec. VIII-C, P32.3-9: "search for occurrences of 64 strings",
//                 "work-group granularity with blocking and weak-ordering"; PAPER.md:30 P30.27-38
//                 grep -F -l).  Each work-group loops over 256 KiB chunks: gsys_pread of the
//                 chunk + halo into its device staging line, then the scan (row a8).
//   scan_kernel   the same scan over text already in HBM (standalone HBM-roofline measurement).
//   bench_kernel  granularity x blocking x ordering microbenchmark (sec. VII).
//
// Scan (reading A9/A10, csrc/scan_core.cuh): a token is a maximal run of [A-Za-z0-9_]; it is owned
// by the chunk that holds its first byte; a dictionary hit is a whole token byte-equal to one of
// <= 64 words of <= 16 bytes.  A warp stages 2 KiB tiles in shared memory (cp.async, double
// buffered); each lane runs its contiguous 64-byte span through a byte DFA built from a trie of the
// dictionary, held transposed in shared memory (one IMAD + one LDS.U16 per byte, no per-token
// divergence); a hit is the entry into a per-word emission state, counted once per byte pair with
// a predicated shared RED into the warp's histogram.  grep tests every owned position whose byte
// is in the first-byte range of the patterns.  No tensor cores: nothing here is a contraction.

#include <cuda.h>
#include <cuda_runtime.h>
#include <errno.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <atomic>
#include <mutex>
#include <vector>

#include "gsys.h"
#include "gsys_device.cuh"
#include "gsys_internal.h"
#include "scan_core.cuh"
#include "tokscan.cuh"

namespace {

using namespace gsys_scan;

struct ScanState {
    const ScanTables* T;        // shared memory: the transposed DFA follows it (DFA scan), or the grep
                                // part of the token tables (token scan)
    const gsys_tok::TokTables* TT;   // shared memory: token tables (token scan) or nullptr
    unsigned* whist;            // this warp's shared histogram [64]
    unsigned char* stage;       // shared memory, WARP_STAGE / TWWARP_STAGE bytes per warp
    int* hit;                   // shared grep-hit flag of the current chunk (nullptr: no grep)
};

// Load policies: LD_NC for text that is immutable during the kernel (HBM scan), LD_CG for device
// staging lines refilled by the copy engine between chunks (L2 is the point of coherence; skip
// L1), LD_SYS for host-mapped staging lines refilled by host preads (ld.cv: cached system-memory
// lines are considered stale and fetched again; unlike strong .sys loads these still coalesce
// into full PCIe read requests -- the strong form ran at ~35 MB/s per work-group).
enum LoadPolicy { LD_NC = 0, LD_CG = 1, LD_SYS = 2, LD_CA = 3 };

template <int P>
__device__ __forceinline__ uint4 ld16(const unsigned char* p) {
    uint4 v;
    if (P == LD_NC)
        asm volatile("ld.global.nc.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    else if (P == LD_CG)
        asm volatile("ld.global.cg.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    else if (P == LD_CA)
        asm volatile("ld.global.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    else
        asm volatile("ld.global.cv.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    return v;
}
template <int P>
__device__ __forceinline__ unsigned ld1(const unsigned char* p) {
    unsigned v;
    if (P == LD_NC) asm volatile("ld.global.nc.u8 %0, [%1];" : "=r"(v) : "l"(p));
    else if (P == LD_CG) asm volatile("ld.global.cg.u8 %0, [%1];" : "=r"(v) : "l"(p));
    else if (P == LD_CA) asm volatile("ld.global.u8 %0, [%1];" : "=r"(v) : "l"(p));
    else asm volatile("ld.global.cv.u8 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v & 0xffu;
}



// Count a DFA entry e if it is an emission (e >= emit2: word (e - emit2) / 2): a predicated shared
// RED at hb + 2 e (hb = histogram address - 2 emit2).  The predicate is set inside the asm, so the
// compiler emits @P RED (no branch, no reconvergence barrier) and lanes without a hit send nothing.
constexpr unsigned HSTRIDE = MAXD + 4;    // per-warp shared words: histogram (+ pad)
__device__ __forceinline__ void red_emit(unsigned hb, unsigned e, unsigned emit2) {
    asm volatile("{ .reg .pred p; setp.ge.u32 p, %1, %2; @p red.shared.add.u32 [%0], 1; }"
                 :: "r"(hb + 2u * e), "r"(e), "r"(emit2) : "memory");
}
// the two pair maxima of a 4-byte group (at most one emission per pair)
__device__ __forceinline__ void red_emit2(unsigned hb, unsigned hi, unsigned lo, unsigned emit2) {
    asm volatile("{ .reg .pred p, q; setp.ge.u32 p, %2, %4; setp.ge.u32 q, %3, %4;\n\t"
                 "@p red.shared.add.u32 [%0], 1; @q red.shared.add.u32 [%1], 1; }"
                 :: "r"(hb + 2u * hi), "r"(hb + 2u * lo), "r"(hi), "r"(lo), "r"(emit2) : "memory");
}

// Scan positions [s, own_end) of a text whose valid bytes end at valid_end; seg0 points at the
// byte of position s (16-byte aligned); seg0[-1] is the byte before s when s > 0.  A warp takes
// 2 KiB tiles.  Each tile arrives by cp.async (LDGSTS: global -> shared without registers, bytes
// past valid_end zero-filled): four coalesced 16 B pieces per lane into a warp-private buffer
// laid out as 33 lane slots of 64 + 16 B (the padding spreads the banks), plus the 16 B after the
// tile and the 4 B word ending at the byte before it.  Two buffers per warp: the copy of tile i+1
// is in flight while the DFA runs over tile i (the PCIe / HBM latency is hidden behind the DFA).
// Lane l then runs the DFA over its contiguous 64 B span with the next slot's first 16 B as
// lookahead.  Every byte crosses the memory system once.
constexpr unsigned SLOT = 80;
constexpr unsigned STAGE_BYTES = 33 * SLOT + 16;       // slots + the 4-byte "previous" word (padded)
constexpr unsigned WARP_STAGE = 2 * STAGE_BYTES;       // double buffer (wc_kernel)
#ifndef GSYS_DFA_NBUF
#define GSYS_DFA_NBUF 1     // staged tiles per warp of the HBM DFA scan (scan_kernel): one tile lets
                            // 32 warps and the 129-column table fit (profiles/r02_dfa32.jsonl)
#endif
#ifndef GSYS_DFA_MAXT
#define GSYS_DFA_MAXT 1024  // scan_kernel threads per block
#endif
constexpr unsigned DWARP_STAGE = GSYS_DFA_NBUF * STAGE_BYTES;

__device__ __forceinline__ void cp_async16(unsigned dst, const void* src, unsigned src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 16, %2;" :: "r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async4(unsigned dst, const void* src, unsigned src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" :: "r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" :: "n"(N) : "memory"); }

// full-size copies (no src-size operand: no zero-fill bookkeeping)
__device__ __forceinline__ void cp_async16_full(unsigned dst, const void* src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" :: "r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async4_full(unsigned dst, const void* src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(dst), "l"(src) : "memory");
}

// issue the copies of the tile starting at `base` into buffer `buf` (shared address)
__device__ __forceinline__ void stage_tile(unsigned buf, const unsigned char* seg0, long long s, long long base,
                                           long long valid_end, unsigned lane) {
    if (base > 0 && base + 2048 + 16 <= valid_end) {   // interior tile: no bounds, no zero fill
        const unsigned char* src = seg0 + (base - s);
        const unsigned d = buf + (lane >> 2) * SLOT + 16u * (lane & 3u);
#pragma unroll
        for (int k = 0; k < 4; k++) cp_async16_full(d + 8u * k * SLOT, src + 512 * k + 16 * lane);
        if (lane == 0u) {
            cp_async16_full(buf + 32u * SLOT, src + 2048);
            cp_async4_full(buf + 33u * SLOT, src - 4);
        }
        return;
    }
#pragma unroll
    for (int k = 0; k < 4; k++) {
        const long long p = base + 512 * k + 16 * lane;
        const long long left = valid_end - p;
        const unsigned n = left >= 16 ? 16u : (left > 0 ? (unsigned)left : 0u);
        const unsigned slot = 8u * k + (lane >> 2);
        cp_async16(buf + slot * SLOT + 16u * (lane & 3u), seg0 + (n ? p - s : 0), n);
    }
    if (lane == 0u) {
        const long long p = base + 2048;
        const long long left = valid_end - p;
        const unsigned n = left >= 16 ? 16u : (left > 0 ? (unsigned)left : 0u);
        cp_async16(buf + 32u * SLOT, seg0 + (n ? p - s : 0), n);
        cp_async4(buf + 33u * SLOT, seg0 + (base > 0 ? base - 4 - s : 0), base > 0 ? 4u : 0u);
    }
}

// NBUF: staged tiles per warp -- 2 (wc_kernel: the next tile's copies, over PCIe in host staging,
// overlap this tile's scan) or 1 (HBM scan: more warps fit, and they cover each other's latency)
template <int P, bool WIDE, unsigned NBUF = 2>
__device__ __forceinline__ void scan_range(const unsigned char* __restrict__ seg0, long long s, long long own_end,
                                           long long valid_end, const ScanState& S) {
    const ScanTables& T = *S.T;
    const Dfa<WIDE> D = dfa_view_shared<WIDE>(T);
    const bool grep = S.hit != nullptr && T.npat > 0;
    const unsigned emit2 = D.emit2;
    const unsigned hb = (unsigned)__cvta_generic_to_shared(S.whist) - 2u * emit2;
    auto emit = [hb, emit2](unsigned e) { red_emit(hb, e, emit2); };
    auto emit2x = [hb, emit2](unsigned hi, unsigned lo) { red_emit2(hb, hi, lo, emit2); };
    const unsigned lane = threadIdx.x & 31u, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    unsigned char* stage = S.stage + warp * NBUF * STAGE_BYTES;
    const unsigned stage_s = (unsigned)__cvta_generic_to_shared(stage);
    const long long step = 2048ll * nwarps;
    long long base = s + 2048ll * warp;
    if (NBUF == 2) {
        if (base < own_end) stage_tile(stage_s, seg0, s, base, valid_end, lane);
        cp_async_commit();
    }
    for (unsigned it = 0; base < own_end; base += step, it ^= (NBUF - 1u)) {
        if (NBUF == 2) {
            const long long nxt = base + step;
            if (nxt < own_end) stage_tile(stage_s + (it ^ 1u) * STAGE_BYTES, seg0, s, nxt, valid_end, lane);
            cp_async_commit();
            cp_async_wait<1>();      // this tile's copies (issued one iteration earlier) have landed
        } else {
            stage_tile(stage_s, seg0, s, base, valid_end, lane);
            cp_async_commit();
            cp_async_wait<0>();
        }
        __syncwarp();
        const unsigned char* buf = stage + it * STAGE_BYTES;
        Win W;
        W.w0 = *reinterpret_cast<const uint4*>(buf + lane * SLOT);
        W.w1 = *reinterpret_cast<const uint4*>(buf + lane * SLOT + 16u);
        W.w2 = *reinterpret_cast<const uint4*>(buf + lane * SLOT + 32u);
        W.w3 = *reinterpret_cast<const uint4*>(buf + lane * SLOT + 48u);
        W.w4 = *reinterpret_cast<const uint4*>(buf + (lane + 1u) * SLOT);
        const unsigned prevb = lane ? (unsigned)buf[(lane - 1u) * SLOT + 63u] : (unsigned)buf[33u * SLOT + 3u];
        const long long p0 = base + 64ll * lane;
        // the block's "a pattern was seen" flag, read once per warp tile (an atomic read, set by
        // atomic writes: the early exit is an optimisation, not a synchronisation)
        const int seen = grep ? __shfl_sync(0xffffffffu, lane == 0u ? atomicOr(S.hit, 0) : 0, 0) : 0;
        if (p0 < own_end) {
            dfa_lane64(D, W, prevb, p0, own_end, valid_end, emit, emit2x);
            if (grep && !seen && grep_lane64(T, W, p0, own_end, valid_end)) atomicExch(S.hit, 1);
        }
        __syncwarp();                // every lane is done with this buffer before it is refilled
    }
    cp_async_wait<0>();
}

// ------------------------------------------------------------------ token-level scan (tokscan.cuh)
// Staging for the token scan: per 2 KiB warp tile, 32 lane slots of 80 B -- the lane's 64 bytes AND
// the 16 bytes after them (a duplicate of the next slot's first 16 B, so a token window starting
// anywhere in the span is contiguous in shared memory) -- then the 4 bytes before the tile.

__device__ __forceinline__ void stage_tile_tok(unsigned buf, const unsigned char* seg0, long long s, long long base,
                                               long long valid_end, unsigned lane) {
    if (base > 0 && base + 2048 + 16 <= valid_end) {   // interior tile: no bounds, no zero fill
        const unsigned char* src = seg0 + (base - s);
        const unsigned d = buf + (lane >> 2) * SLOT + 16u * (lane & 3u);
#pragma unroll
        for (int k = 0; k < 4; k++) cp_async16_full(d + 8u * k * SLOT, src + 512 * k + 16 * lane);
        cp_async16_full(buf + lane * SLOT + 64u, src + 64u * (lane + 1u));
        if (lane == 0u) cp_async4_full(buf + 32u * SLOT, src - 4);
        return;
    }
#pragma unroll
    for (int k = 0; k < 5; k++) {
        const long long p = k < 4 ? base + 512 * k + 16 * lane : base + 64ll * (lane + 1u);
        const unsigned dst = k < 4 ? buf + (8u * k + (lane >> 2)) * SLOT + 16u * (lane & 3u) : buf + lane * SLOT + 64u;
        const long long left = valid_end - p;
        const unsigned n = left >= 16 ? 16u : (left > 0 ? (unsigned)left : 0u);
        cp_async16(dst, seg0 + (n ? p - s : 0), n);
    }
    if (lane == 0u) cp_async4(buf + 32u * SLOT, seg0 + (base > 0 ? base - 4 - s : 0), base > 0 ? 4u : 0u);
}

// Warp-cooperative token scan of positions [s, own_end) (gsys_tok::tokw_*; same contract as
// scan_range; tiles staged by stage_tile_tok): per tile, phase A -- each lane classifies its span, the lanes'
// start counts are prefix-summed with shuffles and every lane appends its entries to the warp's
// list in shared memory; phase C -- lane j looks up entries j, j+32, ... of that list.
#ifndef GSYS_TOK_NBUF
#define GSYS_TOK_NBUF 1     // staged tiles per warp: 1 lets 32 warps fit (their copies cover each
                            // other's latency); 2 overlaps the next tile's copies within a warp
#endif
constexpr unsigned TWWARP_STAGE = GSYS_TOK_NBUF * gsys_tok::TOKW_TILE + 2 * gsys_tok::TOKW_LIST;
// stage_tile_tok fills 32 lane slots and the 4-byte "previous" word at 32 * SLOT; a lookup reads 20
// bytes from its (4-byte aligned) offset, TOKW_SKIP's included
static_assert(SLOT == gsys_tok::TOKW_SLOT && gsys_tok::TOKW_SKIP == 32 * SLOT &&
                  gsys_tok::TOKW_SKIP + 20 <= gsys_tok::TOKW_TILE,
              "the token scan's tile layout must match stage_tile_tok's slots");

__device__ __forceinline__ void scan_range_tokw(const unsigned char* __restrict__ seg0, long long s, long long own_end,
                                                long long valid_end, const ScanState& S) {
    const gsys_tok::TokTables& T = *S.TT;
    const bool grep = S.hit != nullptr && T.g.npat > 0;
    const unsigned lane = threadIdx.x & 31u, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    unsigned char* stage = S.stage + warp * TWWARP_STAGE;
    const unsigned stage_s = (unsigned)__cvta_generic_to_shared(stage);
    const unsigned list_s = stage_s + GSYS_TOK_NBUF * gsys_tok::TOKW_TILE;
    const unsigned hs = (unsigned)__cvta_generic_to_shared(S.whist);
    auto emit = [hs](unsigned d) { asm volatile("red.shared.add.u32 [%0], 1;" :: "r"(hs + 4u * d) : "memory"); };
    gsys_tok::TokRegs R = gsys_tok::tok_regs(T);
    // pin the shared-window addresses in registers (an opaque move: the compiler would otherwise
    // rebuild them from SR_CgaCtaId inside the lookup loop)
    asm volatile("mov.b32 %0, %0;" : "+r"(R.tabs));
    const unsigned one = T.one;
    // grep's first-byte prefilter (grep_lane64): SWAR range constants; g_all -- no prefilter (a
    // pattern starting with a byte >= 0x80)
    const bool g_all = T.g.fb_hi >= 0x80u;
    const unsigned g_add_lo = (0x80u - T.g.fb_lo) * 0x01010101u, g_add_hi = (0x7fu - T.g.fb_hi) * 0x01010101u;
    const long long step = 2048ll * nwarps;
    long long base = s + 2048ll * warp;
#if GSYS_TOK_NBUF == 2
    if (base < own_end) stage_tile_tok(stage_s, seg0, s, base, valid_end, lane);
    cp_async_commit();
#endif
    for (unsigned it = 0; base < own_end; base += step, it ^= (GSYS_TOK_NBUF - 1u)) {
#if GSYS_TOK_NBUF == 2
        const long long nxt = base + step;
        if (nxt < own_end) stage_tile_tok(stage_s + (it ^ 1u) * gsys_tok::TOKW_TILE, seg0, s, nxt, valid_end, lane);
        cp_async_commit();
        cp_async_wait<1>();
#else   // one tile per warp: its copies are waited for at once (other warps cover the latency)
        stage_tile_tok(stage_s, seg0, s, base, valid_end, lane);
        cp_async_commit();
        cp_async_wait<0>();
#endif
        __syncwarp();
        const unsigned char* buf = stage + it * gsys_tok::TOKW_TILE;
        const unsigned buf_s = stage_s + it * gsys_tok::TOKW_TILE;
        const long long p0 = base + 64ll * lane;
        unsigned n;
        {   // phase A
            const unsigned char* span = buf + lane * SLOT;
            Win W;
            W.w0 = *reinterpret_cast<const uint4*>(span);
            W.w1 = *reinterpret_cast<const uint4*>(span + 16u);
            W.w2 = *reinterpret_cast<const uint4*>(span + 32u);
            W.w3 = *reinterpret_cast<const uint4*>(span + 48u);
            W.w4 = *reinterpret_cast<const uint4*>(span + 64u);
            // word-byte masks, with grep's first-byte prefilter fused into the same pass
            unsigned gacc = 0;
            const unsigned m0 = gsys_tok::mask16g(W.w0, one, g_add_lo, g_add_hi, gacc) |
                                (gsys_tok::mask16g(W.w1, one, g_add_lo, g_add_hi, gacc) << 16);
            const unsigned m1 = gsys_tok::mask16g(W.w2, one, g_add_lo, g_add_hi, gacc) |
                                (gsys_tok::mask16g(W.w3, one, g_add_lo, g_add_hi, gacc) << 16);
            unsigned m2 = __shfl_down_sync(0xffffffffu, m0, 1);
            if (lane == 31u) m2 = gsys_tok::mask16(W.w4, one);
            unsigned pw = __shfl_up_sync(0xffffffffu, m1 >> 31, 1);
            if (lane == 0u) pw = base > 0 ? gsys_tok::word4(*reinterpret_cast<const unsigned*>(buf + 32u * SLOT)) >> 31 : 0u;
            // the block's "a pattern was seen" flag, read once per warp tile (an atomic read, set by
            // atomic writes: the early exit is an optimisation, not a synchronisation)
            const int seen = grep ? __shfl_sync(0xffffffffu, lane == 0u ? atomicOr(S.hit, 0) : 0, 0) : 0;
            if (grep && !seen && p0 < own_end && (g_all || (gacc & 0x80808080u)) &&
                grep_lane64_steps(T.g, W, p0, own_end, valid_end))
                atomicExch(S.hit, 1);
            const gsys_tok::TokwSpan sp = gsys_tok::tokw_span(m0, m1, m2, pw != 0u, p0, own_end, valid_end);
            const unsigned cnt = (unsigned)__popc(sp.s0) + (unsigned)__popc(sp.s1);
            unsigned incl = cnt;
#pragma unroll
            for (unsigned d = 1; d < 32u; d <<= 1) {
                const unsigned v = __shfl_up_sync(0xffffffffu, incl, d);
                if (lane >= d) incl += v;
            }
            n = __shfl_sync(0xffffffffu, incl, 31);
            unsigned ptr = list_s + 2u * (incl - cnt);
            gsys_tok::tokw_list(R, sp, lane * SLOT, [&ptr](unsigned e) {
                asm volatile("st.shared.u16 [%0], %1;" :: "r"(ptr), "h"((unsigned short)e) : "memory");
                ptr += 2u;
            });
        }
        __syncwarp();
        {   // phase C
            const gsys_tok::TokwTile tile{buf, buf_s};
            // two entries per round (j, j + 32): their loads are independent, so the lookups'
            // shared-memory latencies overlap (four per round measured slower: registers)
            for (unsigned j = lane; j < n; j += 64u) {
                unsigned e0, e1 = gsys_tok::TOKW_SKIP;
                asm volatile("ld.shared.u16 %0, [%1];" : "=r"(e0) : "r"(list_s + 2u * j) : "memory");
                if (j + 32u < n) asm volatile("ld.shared.u16 %0, [%1];" : "=r"(e1) : "r"(list_s + 2u * j + 64u) : "memory");
                gsys_tok::tokw_lookup(T, R, tile, e0 & 0xffffu, emit);
                gsys_tok::tokw_lookup(T, R, tile, e1 & 0xffffu, emit);
            }
        }
        __syncwarp();                // every lane is done with this buffer and the list before reuse
    }
    cp_async_wait<0>();
}

// ------------------------------------------------------------------ TMA-staged DFA scan (HBM text)
// The same slot layout as stage_tile, filled by the bulk-copy engine instead of per-lane cp.async
// (LDGSTS occupies the LSU pipe the DFA's shared-memory gathers are bound by): lane l copies its
// 64 bytes into slot l, lane 0 the 16 bytes after the tile into slot 32 and the 16 bytes before it
// into the prev area; completion is an mbarrier transaction count per buffer.  Tiles at the ends
// of the text (zero fill, no bytes before position 0) are copied by the lanes themselves.
constexpr unsigned MSTAGE_BYTES = 33 * SLOT + 32;      // slots + 16 B before the tile + the mbarrier
constexpr unsigned MWARP_STAGE = 2 * MSTAGE_BYTES;
constexpr unsigned MPREV = 33 * SLOT;                   // 16 bytes before the tile
constexpr unsigned MBAR = 33 * SLOT + 16;               // 8-byte mbarrier

__device__ __forceinline__ void mbar_init(unsigned bar) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_expect_arrive(unsigned bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" :: "r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned bar, unsigned parity) {
    asm volatile("{\n .reg .pred p;\n WAIT_%=:\n"
                 " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
                 " @!p bra WAIT_%=;\n}" :: "r"(bar), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_copy(unsigned dst, const void* src, unsigned bytes, unsigned bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}

// Stage the tile at `base` into buffer `buf` (shared address); its mbarrier completes either way.
__device__ __forceinline__ void stage_tile_tma(unsigned buf, const unsigned char* seg0, long long s, long long base,
                                               long long valid_end, unsigned lane) {
    const unsigned bar = buf + MBAR;
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // our generic reads of buf come first
    if (base > 0 && base + 2048 + 16 <= valid_end) {
        const unsigned char* src = seg0 + (base - s);
        if (lane == 0u) mbar_expect_arrive(bar, 32u * 64u + 32u);
        __syncwarp();
        bulk_copy(buf + lane * SLOT, src + 64u * lane, 64u, bar);
        if (lane == 0u) {
            bulk_copy(buf + 32u * SLOT, src + 2048, 16u, bar);
            bulk_copy(buf + MPREV, src - 16, 16u, bar);
        }
        return;
    }
    // ends of the text: lanes copy (zero fill past valid_end, nothing before position 0)
    unsigned char* b = reinterpret_cast<unsigned char*>(__cvta_shared_to_generic(buf));
    for (unsigned k = 0; k < 64u; k++) {
        const long long p = base + 64ll * lane + k;
        b[lane * SLOT + k] = p < valid_end ? seg0[p - s] : 0u;
    }
    if (lane < 16u) {
        const long long p = base + 2048 + lane;
        b[32u * SLOT + lane] = p < valid_end ? seg0[p - s] : 0u;
        const long long q = base - 16 + lane;
        b[MPREV + lane] = (q >= 0 && base > 0) ? seg0[q - s] : 0u;
    }
    __syncwarp();
    if (lane == 0u) mbar_arrive(bar);
}

template <bool WIDE>
__device__ __forceinline__ void scan_range_tma(const unsigned char* __restrict__ seg0, long long s, long long own_end,
                                               long long valid_end, const ScanState& S, unsigned& phase) {
    const ScanTables& T = *S.T;
    const Dfa<WIDE> D = dfa_view_shared<WIDE>(T);
    const bool grep = S.hit != nullptr && T.npat > 0;
    const unsigned emit2 = D.emit2;
    const unsigned hb = (unsigned)__cvta_generic_to_shared(S.whist) - 2u * emit2;
    auto emit = [hb, emit2](unsigned e) { red_emit(hb, e, emit2); };
    auto emit2x = [hb, emit2](unsigned hi, unsigned lo) { red_emit2(hb, hi, lo, emit2); };
    const unsigned lane = threadIdx.x & 31u, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    unsigned char* stage = S.stage + warp * MWARP_STAGE;
    const unsigned stage_s = (unsigned)__cvta_generic_to_shared(stage);
    const long long step = 2048ll * nwarps;
    long long base = s + 2048ll * warp;
    if (base < own_end) stage_tile_tma(stage_s, seg0, s, base, valid_end, lane);
    unsigned it = 0;
    for (; base < own_end; base += step, it ^= 1u) {
        const long long nxt = base + step;
        if (nxt < own_end) stage_tile_tma(stage_s + (it ^ 1u) * MSTAGE_BYTES, seg0, s, nxt, valid_end, lane);
        mbar_wait(stage_s + it * MSTAGE_BYTES + MBAR, (phase >> it) & 1u);
        phase ^= 1u << it;
        const unsigned char* buf = stage + it * MSTAGE_BYTES;
        Win W;
        W.w0 = *reinterpret_cast<const uint4*>(buf + lane * SLOT);
        W.w1 = *reinterpret_cast<const uint4*>(buf + lane * SLOT + 16u);
        W.w2 = *reinterpret_cast<const uint4*>(buf + lane * SLOT + 32u);
        W.w3 = *reinterpret_cast<const uint4*>(buf + lane * SLOT + 48u);
        W.w4 = *reinterpret_cast<const uint4*>(buf + (lane + 1u) * SLOT);
        const unsigned prevb = lane ? (unsigned)buf[(lane - 1u) * SLOT + 63u] : (unsigned)buf[MPREV + 15u];
        const long long p0 = base + 64ll * lane;
        // the block's "a pattern was seen" flag, read once per warp tile (an atomic read, set by
        // atomic writes: the early exit is an optimisation, not a synchronisation)
        const int seen = grep ? __shfl_sync(0xffffffffu, lane == 0u ? atomicOr(S.hit, 0) : 0, 0) : 0;
        if (p0 < own_end) {
            dfa_lane64(D, W, prevb, p0, own_end, valid_end, emit, emit2x);
            if (grep && !seen && grep_lane64(T, W, p0, own_end, valid_end)) atomicExch(S.hit, 1);
        }
        __syncwarp();                // every lane is done with this buffer before it is refilled
    }
    (void)it;   // `phase` tracks each buffer's mbarrier parity across ranges
}

// Dynamic shared memory: [tables] [per-warp histograms] [warp stages].  Token tables when tok.
__device__ __forceinline__ unsigned* load_tables_tok(unsigned char* smem, const gsys_tok::TokTables* gT,
                                                     unsigned nwarps, ScanState& S) {
    constexpr size_t tb = (sizeof(gsys_tok::TokTables) + 15) & ~(size_t)15;
    const uint4* src = reinterpret_cast<const uint4*>(gT);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    for (unsigned i = threadIdx.x; i < tb / 16; i += blockDim.x) dst[i] = src[i];
    unsigned* shist = reinterpret_cast<unsigned*>(smem + tb);
    for (unsigned i = threadIdx.x; i < nwarps * HSTRIDE; i += blockDim.x) shist[i] = 0;
    S.stage = smem + tb + nwarps * HSTRIDE * 4;
    S.TT = reinterpret_cast<const gsys_tok::TokTables*>(smem);
    S.T = &S.TT->g;
    S.whist = shist + (threadIdx.x / 32) * HSTRIDE;
    return shist;
}

// Dynamic shared memory: [ScanTables + DFA (tables_bytes)] [per-warp histograms] [warp stages].
__device__ __forceinline__ unsigned* load_tables(unsigned char* smem, const ScanTables* gT, unsigned nwarps,
                                                 ScanState& S) {
    S.TT = nullptr;
    const size_t tb = (tables_bytes(gT->nsp, gT->ncol) + 15) & ~(size_t)15;
    const uint4* src = reinterpret_cast<const uint4*>(gT);
    uint4* dst = reinterpret_cast<uint4*>(smem);
    // DFA entries are rebased to shared addresses (Dfa::org) as they are staged: org + 2 * nsp
    // stays below 64 KiB (the table opens the dynamic window), so each u16 half adds without carry
    static_assert(sizeof(ScanTables) % 16 == 0, "the DFA starts on a 16-byte boundary");
    const unsigned org = (unsigned)__cvta_generic_to_shared(smem) + (unsigned)sizeof(ScanTables);
    const unsigned add = org * 0x10001u;
    for (unsigned i = threadIdx.x; i < tb / 16; i += blockDim.x) {
        uint4 v = src[i];
        if (i >= sizeof(ScanTables) / 16) { v.x += add; v.y += add; v.z += add; v.w += add; }
        dst[i] = v;
    }
    unsigned* shist = reinterpret_cast<unsigned*>(smem + tb);
    for (unsigned i = threadIdx.x; i < nwarps * HSTRIDE; i += blockDim.x) shist[i] = 0;
    S.stage = smem + tb + nwarps * HSTRIDE * 4;
    S.T = reinterpret_cast<const ScanTables*>(smem);
    S.whist = shist + (threadIdx.x / 32) * HSTRIDE;
    return shist;
}

__device__ __forceinline__ void flush_hist(unsigned* shist, unsigned nwarps, unsigned ndict, unsigned long long* hist) {
    for (unsigned d = threadIdx.x; d < ndict; d += blockDim.x) {
        unsigned long long sum = 0;
        for (unsigned w = 0; w < nwarps; w++) sum += shist[w * HSTRIDE + d];
        if (sum) atomicAdd(hist + d, sum);
    }
}

// ------------------------------------------------------------------ wordcount with GPU-issued preads
struct WcArgs {
    const gsys_dev_ctx* ctx;
    const ScanTables* tables;            // DFA scan
    const gsys_tok::TokTables* ttables;  // token scan
    const int* fds;
    const unsigned long long* sizes;
    const unsigned* chunk_base;     // [nfiles + 1] first global chunk of each file
    unsigned char* staging;         // [gridDim.x * stride] host-mapped (host/mixed) or device lines
    unsigned char* staging_dev;     // [gridDim.x * stride] device lines of the mixed mode
    unsigned long long* hist;
    unsigned* file_hits;
    long long* req_ret;
    unsigned long long* prof;       // optional: [0] ns waiting in the call, [1] ns scanning, [2] chunks
    unsigned* next_chunk;           // dynamic chunk queue (zeroed before the launch)
    unsigned nfiles, nchunks, chunk, stride, gflags;
    unsigned host_staging;          // 0 device, 1 host, 2 mixed
    unsigned dev16;                 // mixed: chunks with (k mod 16) < dev16 use the device line
    unsigned prefetch;              // 1: non-blocking preads, two lines per work-group (see below)
};

// One chunk of the global chunk queue: file f, owned range [s, e), request [off, off + len).
struct WcChunk {
    unsigned k, f;
    long long size, s, e, off, len;
};
__device__ __forceinline__ bool wc_next_chunk(const WcArgs& a, unsigned* s_k, WcChunk& c) {
    if (threadIdx.x == 0) *s_k = atomicAdd(a.next_chunk, 1u);
    __syncthreads();
    c.k = *s_k;
    __syncthreads();   // s_k may be overwritten by the next call
    if (c.k >= a.nchunks) return false;
    unsigned lo = 0, hi = a.nfiles;     // largest f with chunk_base[f] <= k
    while (hi - lo > 1) {
        unsigned mid = (lo + hi) >> 1;
        if (a.chunk_base[mid] <= c.k) lo = mid; else hi = mid;
    }
    c.f = lo;
    c.size = (long long)a.sizes[c.f];
    c.s = (long long)(c.k - a.chunk_base[c.f]) * a.chunk;
    c.e = c.s + a.chunk < c.size ? c.s + a.chunk : c.size;
    c.off = c.s ? c.s - 1 : 0;
    c.len = c.e + 16 - c.off;
    return true;
}

template <bool TOK>
__device__ __forceinline__ void scan_line(const unsigned char* seg0, long long s, long long own_end, long long valid_end,
                                          const ScanState& S) {
    if (TOK) scan_range_tokw(seg0, s, own_end, valid_end, S);
    else scan_range<LD_CG, false>(seg0, s, own_end, valid_end, S);
}

template <bool TOK>
__global__ void __launch_bounds__(256, 2) wc_kernel(WcArgs a) {
    // per-chunk grep flag, double-buffered by chunk parity: thread 0 clears the next chunk's flag
    // after reading this one, so no thread can still be touching it (racecheck-clean)
    __shared__ int s_hit[2];
    extern __shared__ __align__(16) unsigned char smem[];
    const unsigned nwarps = blockDim.x / 32;
    ScanState S;
    unsigned* shist = TOK ? load_tables_tok(smem, a.ttables, nwarps, S) : load_tables(smem, a.tables, nwarps, S);
    const ScanTables& sT = *S.T;
    if (threadIdx.x == 0) { s_hit[0] = 0; s_hit[1] = 0; }
    __syncthreads();
    const size_t lines = a.prefetch ? 2u : 1u;
    unsigned char* const hbase = a.staging + (size_t)blockIdx.x * a.stride * lines;
    unsigned char* const dbase = a.host_staging == 2u ? a.staging_dev + (size_t)blockIdx.x * a.stride * lines : hbase;
    unsigned par = 0;
    __shared__ unsigned s_kq;
    if (a.prefetch) {
        // Non-blocking work-group preads, double-buffered (P20.34-46 "non-blocking ... the GPU
        // continues"): the read of the next chunk is issued before this chunk is scanned, and the
        // scan of a line starts after an explicit wait on that read's completion token (slot,
        // seq) -- whatever slot the next call landed in (%smid / %warpid are volatile).  A
        // non-blocking pread returns 0 (A4): the scan takes the bytes a regular file of stable
        // size returns (min(len, size - off)); an error surfaces at gsys_wait.
        __shared__ gsys_token s_tok[2];
        WcChunk c0, c1;
        bool have = wc_next_chunk(a, &s_kq, c0);
        unsigned cur = 0;
        const unsigned nbflags = (a.gflags & ~GSYS_BLOCKING) | GSYS_NONBLOCKING;
        auto line_of = [&](const WcChunk& c, unsigned ln, bool& hostbuf) {
            hostbuf = a.host_staging == 1u || (a.host_staging == 2u && (c.k & 15u) >= a.dev16);
            return (hostbuf ? hbase : dbase) + (size_t)ln * a.stride;
        };
        if (have) {
            bool hb;
            unsigned char* b = line_of(c0, 0, hb);
            const long long r = gsys_pread(a.ctx, a.fds[c0.f], b + 16 - (c0.s - c0.off), (size_t)c0.len, c0.off,
                                           nbflags | (hb ? GSYS_HOSTBUF : 0u), &s_tok[0]);
            if (threadIdx.x == 0 && a.req_ret) a.req_ret[c0.k] = r;
        }
        while (have) {
            const bool more = wc_next_chunk(a, &s_kq, c1);
            if (more) {
                bool hb;
                unsigned char* b = line_of(c1, cur ^ 1u, hb);
                const long long r = gsys_pread(a.ctx, a.fds[c1.f], b + 16 - (c1.s - c1.off), (size_t)c1.len, c1.off,
                                               nbflags | (hb ? GSYS_HOSTBUF : 0u), &s_tok[cur ^ 1u]);
                if (threadIdx.x == 0 && a.req_ret) a.req_ret[c1.k] = r;
            }
            gsys_wait_token(a.ctx, &s_tok[cur], GSYS_WG);   // this line's bytes have landed
            bool hb;
            unsigned char* base = line_of(c0, cur, hb);
            const bool grep = a.file_hits != nullptr && sT.npat > 0 && *(volatile unsigned*)&a.file_hits[c0.f] == 0u;
            const long long valid_end = c0.off + c0.len < c0.size ? c0.off + c0.len : c0.size;
            const long long own_end = c0.e < valid_end ? c0.e : valid_end;
            S.hit = grep ? &s_hit[par] : nullptr;
            if (own_end > c0.s) scan_line<TOK>(base + 16, c0.s, own_end, valid_end, S);
            __syncthreads();   // this line is free for the prefetch issued next iteration
            if (threadIdx.x == 0) {
                if (grep && s_hit[par]) atomicExch(&a.file_hits[c0.f], 1u);
                s_hit[par] = 0;
            }
            par ^= 1u;
            c0 = c1;
            have = more;
            cur ^= 1u;
        }
        __syncthreads();
        flush_hist(shist, nwarps, sT.ndict, a.hist);
        return;
    }
    // Chunks come from a global queue, not a static stride: a work-group takes the next chunk when
    // it is done with its last one, so the ~110 chunk latencies per work-group do not add up into a
    // tail set by the slowest of 296 work-groups.
    __shared__ unsigned s_k;
    for (;;) {
        if (threadIdx.x == 0) s_k = atomicAdd(a.next_chunk, 1u);
        __syncthreads();
        const unsigned k = s_k;
        if (k >= a.nchunks) break;
        unsigned lo = 0, hi = a.nfiles;     // largest f with chunk_base[f] <= k
        while (hi - lo > 1) {
            unsigned mid = (lo + hi) >> 1;
            if (a.chunk_base[mid] <= k) lo = mid; else hi = mid;
        }
        const unsigned f = lo;
        const long long size = (long long)a.sizes[f];
        const long long s = (long long)(k - a.chunk_base[f]) * a.chunk;
        const long long e = s + a.chunk < size ? s + a.chunk : size;
        const long long off = s ? s - 1 : 0;
        const long long len = e + 16 - off;
        // host line (SM zero-copy reads) or device line (copy-engine DMA) for this chunk
        const bool hostbuf = a.host_staging == 1u || (a.host_staging == 2u && (k & 15u) >= a.dev16);
        unsigned char* const base = hostbuf ? hbase : dbase;
        unsigned char* dst = base + 16 - (s - off);
        const bool grep = a.file_hits != nullptr && sT.npat > 0 && *(volatile unsigned*)&a.file_hits[f] == 0u;
        // row a1-a6: one work-group pread of the chunk + halo (P32.7)
        const unsigned long long t0 = a.prof ? gsys::globaltimer() : 0ull;
        const long long r = gsys_pread(a.ctx, a.fds[f], dst, (size_t)len, off,
                                       a.gflags | (hostbuf ? GSYS_HOSTBUF : 0u));
        const unsigned long long t1 = a.prof ? gsys::globaltimer() : 0ull;
        if (threadIdx.x == 0 && a.req_ret) a.req_ret[k] = r;
        if (r > 0) {
            const long long valid_end = off + r;
            const long long own_end = e < valid_end ? e : valid_end;
            S.hit = grep ? &s_hit[par] : nullptr;
            if (own_end > s) scan_line<TOK>(base + 16, s, own_end, valid_end, S);
        }
        __syncthreads();   // the staging line is free again before the next chunk's pread
        if (threadIdx.x == 0) {
            if (grep && s_hit[par]) atomicExch(&a.file_hits[f], 1u);
            s_hit[par] = 0;
        }
        par ^= 1u;
        if (a.prof && threadIdx.x == 0) {
            const unsigned long long t2 = gsys::globaltimer();
            atomicAdd(&a.prof[0], t1 - t0);
            atomicAdd(&a.prof[1], t2 - t1);
            atomicAdd(&a.prof[2], 1ull);
        }
    }
    __syncthreads();
    flush_hist(shist, nwarps, sT.ndict, a.hist);
}

// ------------------------------------------------------------------ scan of HBM-resident text
struct ScanArgs {
    CUtensorMap tmap;               // the text as rows of 64 bytes, 33-row boxes, 64B swizzle (tma_rows > 0)
    const ScanTables* tables;
    const unsigned char* text;
    unsigned long long n;
    unsigned long long* hist;
    unsigned* hit;
    unsigned long long nchunks;
    unsigned chunk;
    unsigned tma_rows;              // full 64-byte rows in the tensor map (0: no tensor-map staging)
};

// ------------------------------------------------------------------ DFA scan with swizzled TMA tiles
// One 2 KiB warp tile (+ the 64-byte row after it) arrives as ONE tensor copy: 33 rows of 64 bytes
// with the hardware 64B swizzle (16-byte chunk c of row r at chunk c ^ ((r >> 1) & 3)), so lane l
// reads row l's chunks (and row l+1's first one) conflict-free with no padding and the staging uses
// no LSU wavefronts.  Tiles that are not whole rows inside the tensor (chunk starts off a 64-byte
// boundary, the text's last partial row) are copied by the lanes into the same swizzled layout,
// zero-filled past valid_end.
constexpr unsigned SW_ROWS = 33, SW_BYTES = SW_ROWS * 64;        // 2112
constexpr unsigned SW_STRIDE = 2560;                               // per warp, keeps 512-B alignment
__device__ __forceinline__ unsigned swz(unsigned row, unsigned chunk) {   // byte offset in a tile
    return row * 64u + 16u * (chunk ^ ((row >> 1) & 3u));
}
__device__ __forceinline__ void stage_tile_swz_lanes(unsigned buf, const unsigned char* seg0, long long s, long long base,
                                                     long long valid_end, unsigned lane) {
    for (unsigned i = lane; i < SW_ROWS * 4u; i += 32u) {
        const unsigned row = i >> 2, c = i & 3u;
        const long long p = base + 64ll * row + 16ll * c;
        const long long left = valid_end - p;
        const unsigned nb = left >= 16 ? 16u : (left > 0 ? (unsigned)left : 0u);
        cp_async16(buf + swz(row, c), seg0 + (nb ? p - s : 0), nb);
    }
}
template <bool WIDE>
__device__ __forceinline__ void scan_range_swz(const ScanArgs& a, const unsigned char* __restrict__ seg0, long long s,
                                               long long own_end, long long valid_end, const ScanState& S,
                                               unsigned char* tiles, unsigned mbar, unsigned& phase) {
    const ScanTables& T = *S.T;
    const Dfa<WIDE> D = dfa_view_shared<WIDE>(T);
    const bool grep = S.hit != nullptr && T.npat > 0;
    const unsigned emit2 = D.emit2;
    const unsigned hb = (unsigned)__cvta_generic_to_shared(S.whist) - 2u * emit2;
    auto emit = [hb, emit2](unsigned e) { red_emit(hb, e, emit2); };
    auto emit2x = [hb, emit2](unsigned hi, unsigned lo) { red_emit2(hb, hi, lo, emit2); };
    const unsigned lane = threadIdx.x & 31u, warp = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    unsigned char* buf = tiles + warp * SW_STRIDE;
    const unsigned buf_s = (unsigned)__cvta_generic_to_shared(buf);
    const long long step = 2048ll * nwarps;
    for (long long base = s + 2048ll * warp; base < own_end; base += step) {
        const bool tma = (base & 63) == 0 && base + 2048 + 64 <= 64ll * a.tma_rows;
        if (tma) {
            if (lane == 0u) {
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(mbar), "r"(SW_BYTES) : "memory");
                asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                             :: "r"(buf_s), "l"(reinterpret_cast<unsigned long long>(&a.tmap)), "r"(0), "r"((int)(base >> 6)),
                                "r"(mbar) : "memory");
            }
            mbar_wait(mbar, phase);
            phase ^= 1u;
        } else {
            stage_tile_swz_lanes(buf_s, seg0, s, base, valid_end, lane);
            cp_async_commit();
            cp_async_wait<0>();
        }
        __syncwarp();
        Win W;
        W.w0 = *reinterpret_cast<const uint4*>(buf + swz(lane, 0));
        W.w1 = *reinterpret_cast<const uint4*>(buf + swz(lane, 1));
        W.w2 = *reinterpret_cast<const uint4*>(buf + swz(lane, 2));
        W.w3 = *reinterpret_cast<const uint4*>(buf + swz(lane, 3));
        W.w4 = *reinterpret_cast<const uint4*>(buf + swz(lane + 1u, 0));
        const long long p0 = base + 64ll * lane;
        unsigned prevb;
        if (lane) prevb = buf[swz(lane - 1u, 3) + 15u];
        else prevb = base > 0 ? (unsigned)__ldg(seg0 + (base - 1 - s)) : 0u;
        const int seen = grep ? __shfl_sync(0xffffffffu, lane == 0u ? atomicOr(S.hit, 0) : 0, 0) : 0;
        if (p0 < own_end) {
            dfa_lane64(D, W, prevb, p0, own_end, valid_end, emit, emit2x);
            if (grep && !seen && grep_lane64(T, W, p0, own_end, valid_end)) atomicExch(S.hit, 1);
        }
        __syncwarp();                // every lane is done with this tile before it is refilled
    }
}

__global__ void __launch_bounds__(GSYS_DFA_MAXT, 1) scan_kernel(const __grid_constant__ ScanArgs a) {
    __shared__ int s_hit;
    __shared__ __align__(8) unsigned long long s_mbar[GSYS_DFA_MAXT / 32];
    extern __shared__ __align__(16) unsigned char smem[];   // tiles aligned at run time (1024 B slack)
    const unsigned nwarps = blockDim.x / 32;
    ScanState S;
    unsigned* shist = load_tables(smem, a.tables, nwarps, S);
    const ScanTables& sT = *S.T;
    const unsigned lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    // tensor-map tiles (a.tma_rows > 0): 1024-aligned per-warp tiles after the histograms
    unsigned char* tiles = reinterpret_cast<unsigned char*>(((uintptr_t)S.stage + 1023) & ~(uintptr_t)1023);
    const unsigned mbar = (unsigned)__cvta_generic_to_shared(&s_mbar[warp]);
    if (a.tma_rows && lane == 0u) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(mbar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (threadIdx.x == 0) s_hit = 0;
    __syncthreads();
    S.hit = a.hit ? &s_hit : nullptr;
    unsigned phase = 0;
    for (unsigned long long k = blockIdx.x; k < a.nchunks; k += gridDim.x) {
        const long long s = (long long)k * a.chunk;
        const long long e = s + a.chunk < (long long)a.n ? s + a.chunk : (long long)a.n;
        if (a.tma_rows) {
            if (sT.ncol == NCOL_WIDE) scan_range_swz<true>(a, a.text + s, s, e, (long long)a.n, S, tiles, mbar, phase);
            else scan_range_swz<false>(a, a.text + s, s, e, (long long)a.n, S, tiles, mbar, phase);
        } else if (sT.ncol == NCOL_WIDE) scan_range<LD_NC, true, GSYS_DFA_NBUF>(a.text + s, s, e, (long long)a.n, S);
        else scan_range<LD_NC, false, GSYS_DFA_NBUF>(a.text + s, s, e, (long long)a.n, S);
    }
    __syncthreads();
    flush_hist(shist, nwarps, sT.ndict, a.hist);
    if (threadIdx.x == 0 && a.hit && s_hit) atomicExch(a.hit, 1u);
}

// The byte-DFA scan with bulk-copy (TMA) staging.
__global__ void __launch_bounds__(768, 1) scan_tma_kernel(ScanArgs a) {
    __shared__ int s_hit;
    extern __shared__ __align__(16) unsigned char smem[];
    const unsigned nwarps = blockDim.x / 32;
    ScanState S;
    unsigned* shist = load_tables(smem, a.tables, nwarps, S);
    const ScanTables& sT = *S.T;
    if (threadIdx.x == 0) s_hit = 0;
    const unsigned lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    if (lane == 0u) {
        const unsigned st = (unsigned)__cvta_generic_to_shared(S.stage + warp * MWARP_STAGE);
        mbar_init(st + MBAR);
        mbar_init(st + MSTAGE_BYTES + MBAR);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    S.hit = a.hit ? &s_hit : nullptr;
    unsigned phase = 0;
    for (unsigned long long k = blockIdx.x; k < a.nchunks; k += gridDim.x) {
        const long long s = (long long)k * a.chunk;
        const long long e = s + a.chunk < (long long)a.n ? s + a.chunk : (long long)a.n;
        if (sT.ncol == NCOL_WIDE) scan_range_tma<true>(a.text + s, s, e, (long long)a.n, S, phase);
        else scan_range_tma<false>(a.text + s, s, e, (long long)a.n, S, phase);
    }
    __syncthreads();
    flush_hist(shist, nwarps, sT.ndict, a.hist);
    if (threadIdx.x == 0 && a.hit && s_hit) atomicExch(a.hit, 1u);
}

// Token-level scan of HBM-resident text (gsys_tok): 1 block of up to 32 warps per SM.
#ifndef GSYS_TOK_MAXT
#define GSYS_TOK_MAXT 1024  // token scan threads per block (register budget 65536 / GSYS_TOK_MAXT)
#endif
__global__ void __launch_bounds__(GSYS_TOK_MAXT, 1) scan_tok_kernel(ScanArgs a) {
    __shared__ int s_hit;
    extern __shared__ __align__(16) unsigned char smem[];
    const unsigned nwarps = blockDim.x / 32;
    ScanState S;
    unsigned* shist = load_tables_tok(smem, reinterpret_cast<const gsys_tok::TokTables*>(a.tables), nwarps, S);
    if (threadIdx.x == 0) s_hit = 0;
    __syncthreads();
    S.hit = a.hit ? &s_hit : nullptr;
    for (unsigned long long k = blockIdx.x; k < a.nchunks; k += gridDim.x) {
        const long long s = (long long)k * a.chunk;
        const long long e = s + a.chunk < (long long)a.n ? s + a.chunk : (long long)a.n;
        scan_range_tokw(a.text + s, s, e, (long long)a.n, S);
    }
    __syncthreads();
    flush_hist(shist, nwarps, S.T->ndict, a.hist);
    if (threadIdx.x == 0 && a.hit && s_hit) atomicExch(a.hit, 1u);
}

// ------------------------------------------------------------------ granularity microbenchmark
struct BenchArgs {
    const gsys_dev_ctx* ctx;
    unsigned char* buf;
    long long* ret;
    unsigned long long* lat;
    unsigned long long* sum;
    unsigned long long len, size;
    int fd;
    unsigned kind, gflags, iters;
};

__device__ __forceinline__ unsigned char pw_byte(unsigned long long idx, unsigned long long i) {
    return (unsigned char)((idx * 131ull + i * 7ull + 13ull) & 0xffull);
}

// Byte sum of buf[0, n) by the threads of the calling scope (WI: the thread alone; WG: the block;
// KERNEL: every block sums the whole region).  Returned to thread 0 of the block (WG/KERNEL).
__device__ unsigned long long scope_sum(const unsigned char* b, unsigned long long n, bool wi) {
    __shared__ unsigned long long s_acc;
    if (wi) {
        unsigned long long acc = 0;
        for (unsigned long long i = 0; i < n; i++) acc += b[i];
        return acc;
    }
    if (threadIdx.x == 0) s_acc = 0;
    __syncthreads();
    unsigned long long acc = 0;
    for (unsigned long long i = threadIdx.x; i < n; i += blockDim.x) acc += b[i];
    atomicAdd(&s_acc, acc);
    __syncthreads();
    unsigned long long r = s_acc;
    __syncthreads();
    return r;
}

__global__ void __launch_bounds__(1024, 1) bench_kernel(BenchArgs a) {   // <= 64 registers: 4 x 256-thread WGs per SM
    const unsigned gran = a.gflags & GSYS_GRAN_MASK;
    const unsigned tid = threadIdx.x;
    const bool wi = gran == GSYS_WI;
    unsigned long long caller;
    bool recorder;
    if (wi) { caller = (unsigned long long)blockIdx.x * blockDim.x + tid; recorder = true; }
    else if (gran == GSYS_WG) { caller = blockIdx.x; recorder = tid == 0; }
    else { caller = 0; recorder = blockIdx.x == 0 && tid == 0; }
    alignas(16) unsigned char ru[160];
    for (unsigned r = 0; r < a.iters; r++) {
        const unsigned long long idx = caller * a.iters + r;
        const unsigned long long off = a.size ? (idx * a.len) % a.size : 0;
        unsigned char* b = a.buf ? a.buf + caller * a.len : nullptr;
        if (a.kind == 2) {
            // produce the payload: every thread of the scope writes its share, late threads first
            // spin, so a call issued without the pre-call barrier would publish stale bytes
            unsigned long long t_end = gsys::globaltimer() + (tid % 7) * 3000ull;
            while (gsys::globaltimer() < t_end) {}
            if (wi) {
                for (unsigned long long i = 0; i < a.len; i++) b[i] = pw_byte(idx, i);
            } else {
                unsigned long long nthr = blockDim.x, start = tid;
                if (gran == GSYS_KERNEL) { nthr *= gridDim.x; start += (unsigned long long)blockIdx.x * blockDim.x; }
                for (unsigned long long i = start; i < a.len; i += nthr) b[i] = pw_byte(idx, i);
            }
        }
        const unsigned long long t0 = gsys::globaltimer();
        long long rv;
        if (a.kind == 0) rv = gsys_getrusage(a.ctx, 0 /* RUSAGE_SELF */, ru, a.gflags);
        else if (a.kind == 1) rv = gsys_pread(a.ctx, a.fd, b, (size_t)a.len, (long long)off, a.gflags);
        else rv = gsys_pwrite(a.ctx, a.fd, b, (size_t)a.len, (long long)off, a.gflags);
        const unsigned long long t1 = gsys::globaltimer();
        unsigned long long sum = 0;
        if (a.kind == 1 && a.sum && !(a.gflags & GSYS_NONBLOCKING)) {
            const unsigned long long n = rv > 0 ? (unsigned long long)rv : 0ull;
            sum = scope_sum(b, n, wi);
        }
        if (recorder) {
            if (a.ret) a.ret[idx] = rv;
            if (a.lat) a.lat[idx] = t1 - t0;
            if (a.kind == 1 && a.sum) a.sum[idx] = sum;
        }
        if (a.kind == 2 && !wi && !(a.gflags & GSYS_NONBLOCKING) && !(a.gflags & GSYS_RELAXED)) {
            // strong consumer: Bar2 already separates the call from the next iteration's writes
        } else if (a.kind == 2) {
            // relaxed consumer: the block waits for its caller before writing the next payload.
            // A non-blocking (or kernel-scope) call has returned before the host read the buffer,
            // so with iters > 1 a later payload may reach the file in its place: those cells
            // measure the call rate; the content checks run them with one call per caller
            __syncthreads();
        }
    }
}

// ------------------------------------------------------------------ host side: tables + workspace
struct Workspace {
    unsigned char* up_h = nullptr;   // pinned upload staging
    unsigned char* up_d = nullptr;
    size_t up_cap = 0;
    cudaEvent_t up_ev = nullptr;
    // recorded after every launch that uses this workspace: a later call -- on any stream -- waits
    // for it on the device before touching the shared chunk queue, uploads or staging lines, so
    // calls on different streams are serialised instead of racing
    cudaEvent_t last_ev = nullptr;
    // the scan tables of the last (dictionary, patterns, implementation, columns) built on the host:
    // building them (trie + DFA fill, or the hash search) costs more CPU time than a config-1 kernel
    // runs, so repeated calls with the same dictionary reuse the blob
    struct TabCache { std::vector<uint8_t> key, blob; unsigned char* d = nullptr; size_t dcap = 0; };
    TabCache tcache[4];
    unsigned tcache_next = 0;
    unsigned char* staging_d = nullptr;
    size_t staging_cap = 0;
    unsigned long long* prof_d = nullptr;  // wc_kernel profile counters (gsys_set_profile)
    unsigned* next_chunk_d = nullptr;      // wc_kernel chunk queue
    bool prof_on = false;
    unsigned char* hstaging = nullptr;    // pinned, host-mapped (zero-copy staging)
    size_t hstaging_cap = 0;
    int sms = 0;
};
Workspace g_ws[64];
std::mutex g_ws_mu;
// scan implementation of wc_kernel / gsys_scan_device: GSYS_SCAN_DFA (default: 1.79 TB/s on the
// 1 GiB HBM scan) or GSYS_SCAN_TOKEN (warp-cooperative token scan, 1.40 TB/s,
// profiles/r02_tokg.jsonl); env GSYS_SCAN=dfa|token at load, gsys_set_scan() at run time
std::atomic<int> g_scan_impl{[] {
    const char* e = getenv("GSYS_SCAN");
    return (e && strcmp(e, "token") == 0) ? (int)GSYS_SCAN_TOKEN
           : (e && strcmp(e, "dfa_tma") == 0) ? (int)GSYS_SCAN_DFA_TMA : (int)GSYS_SCAN_DFA;
}()};

Workspace* workspace() {
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess || d < 0 || d >= 64) return nullptr;
    Workspace* W = &g_ws[d];
    if (!W->up_ev) {
        cudaEventCreateWithFlags(&W->up_ev, cudaEventDisableTiming);
        cudaEventCreateWithFlags(&W->last_ev, cudaEventDisableTiming);
        cudaDeviceGetAttribute(&W->sms, cudaDevAttrMultiProcessorCount, d);
    }
    return W;
}

// The scan tables for (impl, ncol, dictionary, patterns): from the cache, else built.  Returns the
// cache entry (host blob, a 16-byte multiple, and its device copy) or nullptr with *rc set.
Workspace::TabCache* scan_tables(Workspace* W, bool tok, unsigned ncol, const char* dict, const uint8_t* dlen,
                                 uint32_t ndict, const char* pats, const uint8_t* plen, uint32_t npat, int* rc) {
    std::vector<uint8_t> key;
    key.reserve(16 + 18u * (ndict + npat));
    const uint32_t hdr[4] = {tok ? 1u : 0u, ncol, ndict, npat};
    key.insert(key.end(), (const uint8_t*)hdr, (const uint8_t*)hdr + sizeof hdr);
    if (ndict && dict && dlen) {
        key.insert(key.end(), (const uint8_t*)dict, (const uint8_t*)dict + 17ull * ndict);
        key.insert(key.end(), dlen, dlen + ndict);
    }
    if (npat && pats && plen) {
        key.insert(key.end(), (const uint8_t*)pats, (const uint8_t*)pats + 17ull * npat);
        key.insert(key.end(), plen, plen + npat);
    }
    for (auto& c : W->tcache)
        if (!c.blob.empty() && c.key == key) { *rc = 0; return &c; }
    size_t tb = 0;
    int r = tok ? gsys_tok::build_tok_tables(nullptr, 0, dict, dlen, ndict, pats, plen, npat, &tb)
                : build_tables(nullptr, 0, dict, dlen, ndict, pats, plen, npat, &tb, ncol);
    if (r && r != -ENOSPC) { *rc = r; return nullptr; }
    std::vector<uint8_t> blob((tb + 15) & ~(size_t)15, 0);
    r = tok ? gsys_tok::build_tok_tables(blob.data(), blob.size(), dict, dlen, ndict, pats, plen, npat, nullptr)
            : build_tables(blob.data(), blob.size(), dict, dlen, ndict, pats, plen, npat, nullptr, ncol);
    if (r) { *rc = r; return nullptr; }
    auto& c = W->tcache[W->tcache_next++ % 4];
    // the entry's device copy may be in use by a running kernel: wait for the last launch first
    cudaEventSynchronize(W->last_ev);
    if (c.dcap < blob.size()) {
        if (c.d) cudaFree(c.d);
        c.d = nullptr;
        c.dcap = 0;
        if (cudaMalloc((void**)&c.d, blob.size()) != cudaSuccess) { *rc = -ENOMEM; c.blob.clear(); return nullptr; }
        c.dcap = blob.size();
    }
    if (cudaMemcpy(c.d, blob.data(), blob.size(), cudaMemcpyHostToDevice) != cudaSuccess) {
        *rc = -EIO;
        c.blob.clear();
        return nullptr;
    }
    c.key.swap(key);
    c.blob.swap(blob);
    *rc = 0;
    return &c;
}

int ensure_upload(Workspace* W, size_t bytes) {
    cudaEventSynchronize(W->up_ev);   // the previous upload has left the pinned staging
    if (bytes <= W->up_cap) return 0;
    size_t cap = 1 << 16;
    while (cap < bytes) cap <<= 1;
    if (W->up_h) cudaFreeHost(W->up_h);
    if (W->up_d) { cudaDeviceSynchronize(); cudaFree(W->up_d); }
    W->up_h = nullptr; W->up_d = nullptr; W->up_cap = 0;
    if (cudaHostAlloc((void**)&W->up_h, cap, cudaHostAllocDefault) != cudaSuccess) return -ENOMEM;
    if (cudaMalloc((void**)&W->up_d, cap) != cudaSuccess) return -ENOMEM;
    W->up_cap = cap;
    return 0;
}

int ensure_staging(Workspace* W, size_t bytes) {
    if (bytes <= W->staging_cap) return 0;
    if (W->staging_d) { cudaDeviceSynchronize(); cudaFree(W->staging_d); }
    W->staging_d = nullptr; W->staging_cap = 0;
    if (cudaMalloc((void**)&W->staging_d, bytes) != cudaSuccess) return -ENOMEM;
    W->staging_cap = bytes;
    return 0;
}

int ensure_hstaging(Workspace* W, size_t bytes) {
    if (bytes <= W->hstaging_cap) return 0;
    if (W->hstaging) {
        cudaDeviceSynchronize();
        gsys_internal_register_host_range(W->hstaging, W->hstaging_cap, 0);
        cudaFreeHost(W->hstaging);
    }
    W->hstaging = nullptr; W->hstaging_cap = 0;
    if (cudaHostAlloc((void**)&W->hstaging, bytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
        return -ENOMEM;
    W->hstaging_cap = bytes;
    gsys_internal_register_host_range(W->hstaging, bytes, 1);
    return 0;
}

constexpr size_t kSmemDynMax = 227 * 1024 - 64;   // opt-in dynamic shared memory per block (static s_hit aside)

int ensure_smem_attr(const void* fn, size_t bytes) {
    if (bytes <= 48 * 1024) return 0;
    if (bytes > 227 * 1024) return -E2BIG;
    return cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) == cudaSuccess ? 0 : -EINVAL;
}

int map_cuda(cudaError_t e) {
    if (e == cudaSuccess) return 0;
    if (e == cudaErrorMemoryAllocation) return -ENOMEM;
    if (e == cudaErrorInvalidValue || e == cudaErrorInvalidConfiguration) return -EINVAL;
    return -EIO;
}

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

}  // namespace

extern "C" {

int gsys_wordcount(const int32_t* fds, const uint64_t* sizes, uint32_t nfiles, uint32_t chunk, const char* dict,
                   const uint8_t* dlen, uint32_t ndict, const char* pats, const uint8_t* plen, uint32_t npat,
                   uint64_t* d_hist, uint32_t* d_file_hits, int64_t* d_req_ret, uint32_t gflags, uint32_t staging,
                   uint32_t blocks, uint32_t threads, void* stream) {
    gsys_dev_ctx* ctx = gsys_internal_ctx_d();
    if (!ctx) return -ENODEV;
    if ((gflags & GSYS_GRAN_MASK) != GSYS_WG) return -EINVAL;
    const bool prefetch = (gflags & GSYS_NONBLOCKING) != 0;   // non-blocking: double-buffered prefetch
    const size_t nlines = prefetch ? 2 : 1;
    const bool mixed = (staging & ~15u) == GSYS_STAGE_MIXED(0) && (staging & 15u) != 0u;
    if (staging > GSYS_STAGE_HOST && !mixed) return -EINVAL;
    if (nfiles == 0 || !fds || !sizes || (!d_hist && ndict)) return -EINVAL;
    if (chunk < 4096 || (chunk % 16) || chunk > (1u << 30)) return -EINVAL;
    if (threads == 0) threads = 256;
    if (threads % 32 || threads > 256) return -EINVAL;
    std::lock_guard<std::mutex> g(g_ws_mu);
    Workspace* W = workspace();
    if (!W) return -ENODEV;
    // chunk table
    std::vector<unsigned> cbase(nfiles + 1);
    uint64_t nch = 0;
    for (uint32_t f = 0; f < nfiles; f++) {
        cbase[f] = (unsigned)nch;
        nch += (sizes[f] + chunk - 1) / chunk;
        if (nch >= (1ull << 32)) return -EINVAL;
    }
    cbase[nfiles] = (unsigned)nch;
    if (blocks == 0) blocks = 2u * (uint32_t)W->sms;
    if (nch < blocks) blocks = (uint32_t)(nch ? nch : 1);
    // upload: [tables][fds][sizes][cbase]; token tables (default) or the byte DFA (gsys_set_scan)
    const bool tok = g_scan_impl.load() == GSYS_SCAN_TOKEN;
    int rc = 0;
    Workspace::TabCache* tc = scan_tables(W, tok, NCOL_NARROW, dict, dlen, ndict, pats, plen, npat, &rc);
    if (!tc) return rc;
    const size_t tb = tc->blob.size();
    // upload: [fds][sizes][cbase] (the tables are already on the device)
    size_t o_f = 0, o_s = align_up(o_f + 4ull * nfiles, 256),
           o_c = align_up(o_s + 8ull * nfiles, 256), total = align_up(o_c + 4ull * (nfiles + 1), 256);
    rc = ensure_upload(W, total);
    if (rc) return rc;
    memcpy(W->up_h + o_f, fds, 4ull * nfiles);
    memcpy(W->up_h + o_s, sizes, 8ull * nfiles);
    memcpy(W->up_h + o_c, cbase.data(), 4ull * (nfiles + 1));
    cudaStream_t s = (cudaStream_t)stream;
    cudaStreamWaitEvent(s, W->last_ev, 0);
    cudaMemcpyAsync(W->up_d, W->up_h, total, cudaMemcpyHostToDevice, s);
    cudaEventRecord(W->up_ev, s);
    size_t stride = align_up((size_t)chunk + 64, 256);
    unsigned char* stage = nullptr;
    unsigned char* stage_dev = nullptr;
    if (staging == GSYS_STAGE_HOST || mixed) {
        rc = ensure_hstaging(W, stride * blocks * nlines);
        if (rc) return rc;
        cudaHostGetDevicePointer((void**)&stage, W->hstaging, 0);
    }
    if (staging == GSYS_STAGE_DEVICE || mixed) {
        rc = ensure_staging(W, stride * blocks * nlines);
        if (rc) return rc;
        if (mixed) stage_dev = W->staging_d;
        else stage = W->staging_d;
    }
    WcArgs a;
    memset(&a, 0, sizeof a);
    a.ctx = ctx;
    a.tables = reinterpret_cast<const ScanTables*>(tc->d);
    a.ttables = reinterpret_cast<const gsys_tok::TokTables*>(tc->d);
    a.fds = reinterpret_cast<const int*>(W->up_d + o_f);
    a.sizes = reinterpret_cast<const unsigned long long*>(W->up_d + o_s);
    a.chunk_base = reinterpret_cast<const unsigned*>(W->up_d + o_c);
    a.staging = stage;
    a.staging_dev = stage_dev;
    if (W->prof_on) {
        if (!W->prof_d && cudaMalloc((void**)&W->prof_d, 64) != cudaSuccess) return -ENOMEM;
        a.prof = W->prof_d;
    }
    a.host_staging = mixed ? 2u : (staging == GSYS_STAGE_HOST ? 1u : 0u);
    a.dev16 = mixed ? (staging & 15u) : 0u;
    a.prefetch = prefetch ? 1u : 0u;
    a.hist = reinterpret_cast<unsigned long long*>(d_hist);
    a.file_hits = d_file_hits;
    a.req_ret = reinterpret_cast<long long*>(d_req_ret);
    if (!W->next_chunk_d && cudaMalloc((void**)&W->next_chunk_d, 256) != cudaSuccess) return -ENOMEM;
    a.next_chunk = W->next_chunk_d;
    a.nfiles = nfiles;
    a.nchunks = (unsigned)nch;
    a.chunk = chunk;
    a.stride = (unsigned)stride;
    a.gflags = gflags & ~GSYS_NONBLOCKING;   // the blocking flavour; prefetch derives the rest
    if (nch == 0) return 0;
    void* args[] = {&a};
    const void* fn = tok ? (const void*)wc_kernel<true> : (const void*)wc_kernel<false>;
    size_t smem = align_up(tb, 16) + (threads / 32) * (HSTRIDE * 4 + (tok ? TWWARP_STAGE : WARP_STAGE));
    rc = ensure_smem_attr(fn, smem);
    if (rc) return rc;
    if (cudaMemsetAsync(W->next_chunk_d, 0, 4, s) != cudaSuccess) return -EIO;
    rc = gsys_internal_launch(fn, blocks, threads, args, smem, stream, false);   // no kernel-scope calls
    cudaEventRecord(W->last_ev, s);
    return rc;
}

int gsys_set_profile(int on) {
    std::lock_guard<std::mutex> g(g_ws_mu);
    Workspace* W = workspace();
    if (!W) return -ENODEV;
    W->prof_on = on != 0;
    if (W->prof_on && !W->prof_d) {
        if (cudaMalloc((void**)&W->prof_d, 64) != cudaSuccess) return -ENOMEM;
        cudaMemset(W->prof_d, 0, 64);
    }
    return 0;
}

int gsys_read_profile(uint64_t* out3, int reset) {
    std::lock_guard<std::mutex> g(g_ws_mu);
    Workspace* W = workspace();
    if (!W || !W->prof_d) return -ENODEV;
    if (cudaMemcpy(out3, W->prof_d, 24, cudaMemcpyDeviceToHost) != cudaSuccess) return -EIO;
    if (reset) cudaMemset(W->prof_d, 0, 64);
    return 0;
}

}  // extern "C" (reopened below)

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link dependency)
typedef CUresult (*PFN_tmap_t)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                               const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                               CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static PFN_tmap_t tmap_encoder() {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn) {
        cudaGetLastError();
        return nullptr;
    }
    return (PFN_tmap_t)fn;
}
static bool swz_enabled() {
    static const bool on = [] {
        const char* e = getenv("GSYS_SCAN_SWZ");
        return !(e && strcmp(e, "0") == 0);
    }();
    return on;
}

extern "C" {

int gsys_set_scan(int impl) {
    if (impl != (int)GSYS_SCAN_TOKEN && impl != (int)GSYS_SCAN_DFA && impl != (int)GSYS_SCAN_DFA_TMA) return -EINVAL;
    return g_scan_impl.exchange(impl);
}

int gsys_scan_device(const uint8_t* d_text, uint64_t n, uint32_t chunk, const char* dict, const uint8_t* dlen,
                     uint32_t ndict, const char* pats, const uint8_t* plen, uint32_t npat, uint64_t* d_hist,
                     uint32_t* d_hit, uint32_t blocks, uint32_t threads, void* stream) {
    if ((!d_hist && ndict) || (n && !d_text)) return -EINVAL;
    if (chunk < 16 || chunk % 16) return -EINVAL;
    if ((uintptr_t)d_text % 16) return -EINVAL;
    const int impl = g_scan_impl.load();
    const bool tok = impl == GSYS_SCAN_TOKEN;
    // DFA: 32 warps with one staged tile each + the 129-column table (profiles/r02_dfa32.jsonl:
    // 1.67 TB/s against 1.48 for 24 double-buffered warps + the 77-column one); token: 32
    // warps (one staged tile + a 2 KiB start list per warp; profiles/r02_tokbuf2.jsonl)
    if (threads == 0) threads = impl == GSYS_SCAN_DFA_TMA ? 704 : 1024;
    if (threads % 32 || threads > (tok ? (unsigned)GSYS_TOK_MAXT : impl == GSYS_SCAN_DFA_TMA ? 768u : (unsigned)GSYS_DFA_MAXT)) return -EINVAL;
    std::lock_guard<std::mutex> g(g_ws_mu);
    Workspace* W = workspace();
    if (!W) return -ENODEV;
    // DFA: the 129-column table when it fits next to the warps' staging (1 block of `threads` per
    // SM), else the 77-column one
    int rc = 0;
    Workspace::TabCache* tc = scan_tables(W, tok, NCOL_WIDE, dict, dlen, ndict, pats, plen, npat, &rc);
    if (!tc) return rc;
    // bulk-copy (TMA) staging: measured 1.13-1.17 TB/s vs 1.46 with per-lane cp.async
    // (profiles/r02_scan_staging_ab.jsonl: 33 small bulk copies per 2 KiB tile cost more than the
    // LSU slots they free), so it is the opt-in GSYS_SCAN_DFA_TMA
    const bool tma = impl == GSYS_SCAN_DFA_TMA;
    // the default DFA stages its tiles by one swizzled tensor copy each (scan_range_swz) when the
    // text holds at least one tile of whole 64-byte rows (env GSYS_SCAN_SWZ=0: per-lane cp.async)
    ScanArgs a;
    memset(&a, 0, sizeof a);
    if (!tok && !tma && n / 64 >= SW_ROWS && swz_enabled()) {
        static PFN_tmap_t enc = tmap_encoder();
        const cuuint64_t dims[2] = {64, n / 64};
        const cuuint64_t strides[1] = {64};
        const cuuint32_t box[2] = {64, SW_ROWS};
        const cuuint32_t estr[2] = {1, 1};
        if (enc && enc(&a.tmap, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, const_cast<uint8_t*>(d_text), dims, strides, box,
                       estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B,
                       CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS)
            a.tma_rows = (unsigned)(n / 64);
    }
    const size_t per_warp = HSTRIDE * 4 + (tok ? TWWARP_STAGE : tma ? MWARP_STAGE : a.tma_rows ? SW_STRIDE : DWARP_STAGE);
    const size_t slack = a.tma_rows ? 1024 : 0;   // the tiles start on a 1024-byte boundary
    if (!tok && tc->blob.size() + (threads / 32) * per_warp + slack > kSmemDynMax) {
        tc = scan_tables(W, tok, NCOL_NARROW, dict, dlen, ndict, pats, plen, npat, &rc);
        if (!tc) return rc;
    }
    const size_t tb = tc->blob.size();
    cudaStream_t s = (cudaStream_t)stream;
    cudaStreamWaitEvent(s, W->last_ev, 0);
    unsigned long long nch = (n + chunk - 1) / chunk;
    if (nch == 0) return 0;
    const bool blocks_auto = blocks == 0;
    if (blocks == 0) blocks = (uint32_t)W->sms;
    if (nch < blocks) blocks = (uint32_t)nch;
    a.tables = reinterpret_cast<const ScanTables*>(tc->d);
    a.text = d_text;
    a.n = n;
    a.hist = reinterpret_cast<unsigned long long*>(d_hist);
    a.hit = d_hit;
    a.nchunks = nch;
    a.chunk = chunk;
    const void* fn = tok ? (const void*)scan_tok_kernel : tma ? (const void*)scan_tma_kernel : (const void*)scan_kernel;
    size_t smem = align_up(tb, 16) + (threads / 32) * per_warp + slack;
    rc = ensure_smem_attr(fn, smem);
    if (rc) return rc;
    if (blocks_auto) {   // one full wave: resident blocks per SM x SMs
        int per_sm = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, (int)threads, smem) != cudaSuccess ||
            per_sm < 1)
            per_sm = 1;
        blocks = (uint32_t)per_sm * (uint32_t)W->sms;
        if (nch < blocks) blocks = (uint32_t)nch;
    }
    void* args[] = {&a};
    rc = map_cuda(cudaLaunchKernel(fn, dim3(blocks), dim3(threads), args, smem, s));
    cudaEventRecord(W->last_ev, s);
    return rc;
}

int gsys_bench_calls(uint32_t kind, uint32_t gflags, uint32_t blocks, uint32_t threads, uint32_t iters, int32_t fd,
                     uint64_t len, uint64_t size, void* d_buf, int64_t* d_ret, uint64_t* d_lat_ns, uint64_t* d_sum,
                     void* stream) {
    gsys_dev_ctx* ctx = gsys_internal_ctx_d();
    if (!ctx) return -ENODEV;
    if (kind > 2 || blocks == 0 || threads == 0 || threads > 1024 || iters == 0) return -EINVAL;
    if (kind >= 1 && (size == 0 || len == 0 || !d_buf)) return -EINVAL;
    BenchArgs a;
    memset(&a, 0, sizeof a);
    a.ctx = ctx;
    a.buf = (unsigned char*)d_buf;
    a.ret = reinterpret_cast<long long*>(d_ret);
    a.lat = reinterpret_cast<unsigned long long*>(d_lat_ns);
    a.sum = reinterpret_cast<unsigned long long*>(d_sum);
    a.len = len;
    a.size = size ? size : 1;
    a.fd = fd;
    a.kind = kind;
    a.gflags = gflags;
    a.iters = iters;
    void* args[] = {&a};
    int rc = gsys_launch((const void*)bench_kernel, blocks, 1, 1, threads, 1, 1, args, 0, stream);
    if (rc) return rc;
    unsigned g = gflags & GSYS_GRAN_MASK;
    return g == GSYS_WI ? (int)(blocks * threads) : g == GSYS_WG ? (int)blocks : 1;
}

}  // extern "C"
