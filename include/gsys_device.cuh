/*
 * gsys_device.cuh -- device side of libgsys (sm_100a): GPU-issued POSIX system calls.
 *
 * Implements, per GPU thread, the invocation half of GENESYS (sec. VI):
 *   a1 caller election + pre-call barrier    P22.39-42, P20.14-33
 *   a2 slot claim (cmp-swap, "delayed" if not free)                    P24.10-11, P24.46
 *   a3 marshal nr/flags/seq/args into the 64 B slot (128-bit stores)   P24.8-13
 *   a4 publish (__threadfence_system) + doorbell (the s_sendmsg analogue, warp-aggregated)
 *                                                                       P24.12-14, P16.0
 *   a5 blocking: poll the completion word with backoff; non-blocking: return at once
 *                                                                       P24.15, P24.32-36
 *   a6 post-call barrier + result broadcast                             P22.41-42, P28.2-3
 *
 * B200 mapping: the syscall area, doorbell ring, completion words `hdone` and
 * the pull areas live in pinned host-mapped memory (posted PCIe writes from the GPU, cache-resident
 * for the host); the claim words and per-slot sequence numbers live in device memory, so GPU-GPU
 * arbitration (atomicCAS) stays in L2 (Table-IV analogue: a cmp-swap costs ~0.4 us there, ~1.2 us
 * on host memory).  The host completes a request by storing {seq, ret} into `hdone` after the
 * result (and any pulled bytes) -- the caller's acquire load of its seq makes them visible; the
 * alternative copy-engine paths complete through `mirror` (stream memop) or `hdone` after the DMA.
 * Device-buffer preads are pulled by the caller out of host-mapped memory (B12/B13), non-blocking
 * ones deferred until a token wait, the slot's next claim or gsys_wait (B15).
 *
 * Usage: every device function takes the instance context `const gsys_dev_ctx*` (from
 * gsys_device_ctx()).  Calls of WG granularity must be reached by every thread of the block,
 * calls of KERNEL granularity by every thread of every block (reading A16).  Non-blocking calls
 * may hand back a `gsys_token` (trailing argument) for gsys_wait_token().  Every wait on the host is
 * bounded by the instance's watchdog (-ETIMEDOUT, gsys_set_poll_timeout).
 */
#ifndef GSYS_DEVICE_CUH
#define GSYS_DEVICE_CUH

#include <cuda_runtime.h>
#include <errno.h>
#include <stdint.h>

#include "gsys.h"

#define GSYS_KSITES GSYS_KSITES_MAX   /* kernel-scope call sites per launch (gsys.h)  */
#define GSYS_KROUNDS 4096u      /* kernel-scope calls per site per launch      */

/* Per (site, round) record of a kernel-scope call (reset by gsys_launch). */
struct gsys_kround {
    unsigned arrive;   /* blocks that reached this round of the site            */
    unsigned done;     /* 1 once the caller stored ret (producer calls)          */
    long long ret;     /* the caller's result, broadcast to the other blocks     */
};

/* Watchdog log (device memory, written by the GPU, read and cleared by gsys_wait): every wait that
 * ran out of time (ctx->poll_timeout_ns) bumps `count` and, for the first GSYS_WD_RECS, records
 * which slot / request / call it was and in which phase.  The slot stays claimed (poisoned) until
 * gsys_wait has drained the service, then it is returned to free. */
#define GSYS_WD_RECS 64u
enum gsys_wd_phase { GSYS_WD_CLAIM = 1, GSYS_WD_NBPEND = 2, GSYS_WD_COMPLETION = 3, GSYS_WD_KERNEL = 4,
                     GSYS_WD_TOKEN = 5 };
struct gsys_wd_log {
    unsigned count;
    unsigned pad;
    struct { unsigned slot, seq, nr, phase; } rec[GSYS_WD_RECS];
};

/* Deferred pull of a non-blocking pread into device memory (reading B15): the service reads into
 * a host-mapped range and records it here, at the request's doorbell-ring position; whoever needs
 * the bytes -- a gsys_wait_token() on the request, or gsys_wait()'s flush kernel -- copies them to
 * dst and sets `consumed`, which recycles the range.  tag = position + 1 once written. */
struct gsys_nbrec {
    unsigned long long src;   /* device address of the host-mapped range, 0: nothing to copy */
    unsigned long long dst;
    long long ret;            /* pread result: bytes to copy when > 0                        */
    unsigned tag;
    unsigned consumed;        /* written 1 by the copier (GPU or flush kernel)                */
};

/* Instance context in device memory (built by gsys_init). */
struct gsys_dev_ctx {
    gsys_slot* area;                /* host-mapped [nslots] syscall area                    */
    unsigned char* inline_buf;      /* host-mapped [nslots * GSYS_INLINE_BYTES]             */
    unsigned* claim;                /* device [nslots]: 0 free, 1 owned                     */
    unsigned* seqs;                 /* device [nslots]: last sequence number used           */
    unsigned long long* mirror;     /* device [nslots]: completion word (seq << 32 | u32 ret) */
    unsigned long long* hdone;      /* host-mapped [nslots]: completion word for host-store completions */
    unsigned* lat_hint;             /* device [nslots]: learned sleep before the first host poll (ns) */
    unsigned* nbpend;               /* device [nslots]: seq of a non-blocking request still in service */
    unsigned long long* ring;       /* host-mapped [ring_mask+1] doorbell entries           */
    unsigned* ring_tail;            /* device: next doorbell position                       */
    gsys_kround* krounds;           /* device [GSYS_KSITES * GSYS_KROUNDS]                  */
    unsigned* kblock;               /* device [kblock_cap * GSYS_KSITES]: rounds per block  */
    gsys_trace_rec* trace;          /* device trace buffer or nullptr                       */
    unsigned* trace_n;
    unsigned trace_cap;
    unsigned kblock_cap;
    unsigned nslots;
    unsigned ring_mask;
    unsigned poll_ns_max;           /* backoff cap for device-memory polls                      */
    unsigned poll_ns_host;          /* poll interval for host-memory (PCIe) polls               */
    unsigned pull_big_bytes;        /* pull area of each slot s with s % 32 == 0 (0: none)      */
    unsigned char* pull_big;        /* host-mapped [(nslots / 32) * pull_big_bytes]            */
    unsigned no_hint;               /* 1: no learned pre-poll sleep (env GSYS_SLEEP_HINT=0)     */
    unsigned long long* diag;       /* device [8] phase accumulators (env GSYS_DIAG_PHASES=1) or null */
    unsigned memop_completion;      /* 1 (default): DMA'd blocking calls complete by a stream
                                       memop into `mirror`; 0 (env GSYS_COMPLETION=host): by a
                                       host store into `hdone` once the DMA has drained          */
    unsigned pull_bounce;           /* 1: blocking work-group preads into device memory that fit no
                                       pull area are read into the service's host-mapped bounce
                                       and copied by the work-group (no CUDA call in the service;
                                       env GSYS_COMPLETION=pull)                                  */
    unsigned long long poll_timeout_ns;  /* watchdog: a claim or completion wait longer than this
                                       returns -ETIMEDOUT (0 = wait forever)                      */
    gsys_wd_log* wd;                /* device: watchdog log                                       */
    gsys_nbrec* nbrec;              /* host-mapped [ring_mask+1]: deferred-pull records (B15)     */
    unsigned* nbpos;                /* device [nslots]: ring position of the slot's last non-blocking request */
    unsigned* nbclaim;              /* device [ring_mask+1]: position + 1 of the record whose copy is claimed */
};

/* Explicit completion token of a non-blocking call (slot, seq, ring position): gsys_wait_token()
 * waits for that request whatever slot the caller's next call lands in (%smid / %warpid are
 * volatile), and finishes its deferred pull if it has one. */
struct gsys_token {
    unsigned slot;
    unsigned seq;    /* 0: no request outstanding */
    unsigned pos;    /* the request's doorbell-ring position: names its deferred-pull record */
    unsigned pad_;
};

#ifdef __CUDACC__
namespace gsys {

/* Small per-call payloads carried in the slot's host-mapped inline line (GSYS_INLINE_BYTES):
 * `in` is copied there by the caller before the request is published (siginfo, sockaddr), `out`
 * receives the host's result after a blocking call completes (struct rusage). */
struct InlineIO {
    void* out = nullptr;
    unsigned out_bytes = 0;
    const void* in = nullptr;
    unsigned in_bytes = 0;
};

/* ------------------------------------------------------------------ PTX helpers */
__device__ __forceinline__ unsigned smid() { unsigned r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }
__device__ __forceinline__ unsigned warpid() { unsigned r; asm volatile("mov.u32 %0, %%warpid;" : "=r"(r)); return r; }
__device__ __forceinline__ unsigned laneid() { unsigned r; asm volatile("mov.u32 %0, %%laneid;" : "=r"(r)); return r; }
__device__ __forceinline__ unsigned lanemask_lt() { unsigned r; asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(r)); return r; }
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t;
}
__device__ __forceinline__ unsigned long long ld_relaxed_sys(const unsigned long long* p) {
    unsigned long long v; asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned* p) {
    unsigned v; asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory"); return v;
}
__device__ __forceinline__ void st_relaxed_sys(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" :: "l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned cas_acquire_gpu(unsigned* p, unsigned cmp, unsigned v) {
    unsigned old;
    asm volatile("atom.acquire.gpu.global.cas.b32 %0, [%1], %2, %3;" : "=r"(old) : "l"(p), "r"(cmp), "r"(v) : "memory");
    return old;
}
__device__ __forceinline__ void st_release_gpu(unsigned* p, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" :: "l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_v4_sys(void* p, uint4 v) {
    asm volatile("st.relaxed.sys.global.v4.u32 [%0], {%1, %2, %3, %4};"
                 :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ uint4 ld_v4_sys(const uint4* p) {
    uint4 v;
    asm volatile("ld.relaxed.sys.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    return v;
}
/* Weak 16-byte load of a host-written result.  Used only after the caller's acquire of the
 * completion word (ld.acquire.sys, which also invalidates this SM's L1) -- or, for the other
 * threads of a work-group, after the Bar2 barrier that follows it -- so by the PTX memory model it
 * observes everything the host wrote before its release store.  Weak loads of one thread are
 * pipelined; strong .sys (or .cv) loads are issued one round trip at a time (a 144 B rusage cost
 * 5 us that way, profiles/r01_phase_probe.jsonl). */
__device__ __forceinline__ uint4 ld_v4_after_acquire(const uint4* p) {
    uint4 v;
    asm volatile("ld.global.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p) : "memory");
    return v;
}
#ifdef GSYS_POLL_RELAXED_FENCE
#define GSYS_POLL_LOAD ld_relaxed_sys
#else
#define GSYS_POLL_LOAD ld_acquire_sys
#endif
__device__ __forceinline__ void fence_acq_rel_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }
__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
    unsigned long long v; asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory"); return v;
}

__device__ __forceinline__ unsigned block_tid() {
    return threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
}
__device__ __forceinline__ unsigned block_threads() { return blockDim.x * blockDim.y * blockDim.z; }
__device__ __forceinline__ unsigned block_linear() {
    return blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
}

/* ------------------------------------------------------------------ tracing (debug)
 * One record per slot transition (gsys.h gsys_trace_rec), stamped with %globaltimer where the
 * transition becomes visible: callers stamp after the observation an edge depends on and before
 * the store that hands the slot on. */
__device__ __forceinline__ void trace(const gsys_dev_ctx* c, unsigned s, unsigned seq, unsigned from,
                                      unsigned to, bool blocking, unsigned nr) {
    if (c->trace == nullptr) return;
    const unsigned long long t = globaltimer();
    unsigned i = atomicAdd(c->trace_n, 1u);
    if (i < c->trace_cap) {
        gsys_trace_rec r;
        r.slot = s; r.seq = seq; r.from = (uint8_t)from; r.to = (uint8_t)to; r.actor = 0;
        r.blocking = blocking ? 1 : 0; r.nr = nr; r.t_ns = t;
        c->trace[i] = r;
    }
}

/* ------------------------------------------------------------------ watchdog
 * Every wait on another agent is bounded by ctx->poll_timeout_ns: a lost completion must not hang
 * the GPU (PAPER.md:30 P30.0, GPU timeouts kill the application; PAPER.md:22 P22.0, a failed
 * blocking call should "raise an alarm").  The expired wait is logged in the host-mapped log and
 * the call returns -ETIMEDOUT; gsys_wait() reports it. */
__device__ __forceinline__ bool expired(const gsys_dev_ctx* c, unsigned long long& t0) {
    if (c->poll_timeout_ns == 0ull) return false;
    const unsigned long long t = globaltimer();
    if (t0 == 0ull) { t0 = t; return false; }
    return t - t0 > c->poll_timeout_ns;
}
__device__ __forceinline__ void wd_log(const gsys_dev_ctx* c, unsigned s, unsigned seq, unsigned nr, unsigned phase) {
    if (c->wd == nullptr) return;
    const unsigned i = atomicAdd(&c->wd->count, 1u);
    if (i < GSYS_WD_RECS) {
        c->wd->rec[i].slot = s; c->wd->rec[i].seq = seq; c->wd->rec[i].nr = nr; c->wd->rec[i].phase = phase;
    }
}

/* ------------------------------------------------------------------ a2: claim
 * The slot is chosen by the hardware ID of the calling thread (SM, hardware warp slot, lane),
 * not the programmer-visible ID (PAPER.md:24 P24.2-6; reading A5).  Exclusivity comes from the
 * cmp-swap on the device claim word (P24.46), so a stale %warpid can never double-book a slot;
 * "If the slot is not free, system call invocation is delayed" (P24.11): spin with backoff. */
__device__ __forceinline__ unsigned hw_slot(const gsys_dev_ctx* c) {
    return ((smid() * 64u + warpid()) * 32u + laneid()) % c->nslots;
}

constexpr unsigned NOSLOT = 0xffffffffu;

/* One thread copies r bytes of a host-mapped area (16-byte aligned) to dst: eight 16-byte loads in
 * flight per round trip over PCIe. */
__device__ __forceinline__ void pull_copy_thread(const unsigned char* src, unsigned char* dst, long long r);

/* Exactly one GPU copier per deferred pull (a token wait, the slot's next claim, gsys_wait's
 * flush kernel may all find it pending): the winner of this device-memory cmp-swap copies; the
 * others wait until it is consumed (so their caller can rely on the bytes). */
__device__ __forceinline__ bool claim_record(const gsys_dev_ctx* c, unsigned pos) {
    unsigned* w = c->nbclaim + (pos & c->ring_mask);
    unsigned old = *(volatile unsigned*)w;
    while (old != pos + 1u) {
        const unsigned prev = atomicCAS(w, old, pos + 1u);
        if (prev == old) return true;
        old = prev;
    }
    return false;
}
__device__ __forceinline__ void wait_consumed(const gsys_dev_ctx* c, const gsys_nbrec* q) {
    unsigned long long t0 = 0ull;
    const unsigned long long* w = reinterpret_cast<const unsigned long long*>(&q->tag);   /* {tag, consumed} */
    while ((unsigned)(ld_acquire_sys(w) >> 32) == 0u) {
        __nanosleep(c->poll_ns_host);
        if (expired(c, t0)) return;
    }
}

/* The slot's previous non-blocking request, if it left a small (<= 16 KiB) deferred pull nobody has
 * consumed: waits for its completion word (bounded) and returns its record, claimed for the
 * caller's scope to copy, else nullptr (nothing pending, or another copier had it: then it has
 * landed). */
__device__ __forceinline__ const gsys_nbrec* small_deferred_pending(const gsys_dev_ctx* c, unsigned s) {
    const unsigned pend = c->nbpend[s];
    if (!pend) return nullptr;
    unsigned long long t0 = 0ull;
    while ((unsigned)(ld_acquire_sys(c->hdone + s) >> 32) != pend) {
        __nanosleep(c->poll_ns_host);
        if (expired(c, t0)) return nullptr;   // claim() logs it
    }
    const unsigned pos = c->nbpos[s];
    const gsys_nbrec* q = c->nbrec + (pos & c->ring_mask);
    const uint4 t = ld_v4_after_acquire(reinterpret_cast<const uint4*>(q) + 1);   /* {ret, tag, consumed} */
    const long long r = (long long)((unsigned long long)t.x | ((unsigned long long)t.y << 32));
    if (t.z != pos + 1u || t.w != 0u || r <= 0 || r > 16384) return nullptr;
    const uint4 h = ld_v4_after_acquire(reinterpret_cast<const uint4*>(q));
    if ((h.x | h.y) == 0u) return nullptr;
    if (claim_record(c, pos)) return q;
    wait_consumed(c, q);
    return nullptr;
}

/* The deferred pull at ring position pos, if it is still pending and small (<= 16 KiB): this thread
 * copies it and marks it consumed (the record was written before the completion word this thread
 * has acquired). */
__device__ __forceinline__ void consume_small_deferred(const gsys_dev_ctx* c, unsigned pos) {
    gsys_nbrec* q = c->nbrec + (pos & c->ring_mask);
    const uint4 t = ld_v4_after_acquire(reinterpret_cast<const uint4*>(q) + 1);   /* {ret, tag, consumed} */
    const long long r = (long long)((unsigned long long)t.x | ((unsigned long long)t.y << 32));
    if (t.z != pos + 1u || t.w != 0u || r <= 0 || r > 16384) return;
    const uint4 h = ld_v4_after_acquire(reinterpret_cast<const uint4*>(q));
    if ((h.x | h.y) == 0u) return;
    if (!claim_record(c, pos)) { wait_consumed(c, q); return; }
    pull_copy_thread(reinterpret_cast<const unsigned char*>((unsigned long long)h.x | ((unsigned long long)h.y << 32)),
                     reinterpret_cast<unsigned char*>((unsigned long long)h.z | ((unsigned long long)h.w << 32)), r);
    asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(&q->consumed), "r"(1u) : "memory");
}

__device__ __forceinline__ unsigned claim(const gsys_dev_ctx* c, unsigned nr) {
    unsigned s = hw_slot(c);
    unsigned ns = 32;
    unsigned long long t0 = 0ull;
    /* cmp-swap with acquire semantics: the slot's previous owner's writes (seqs[s], nbpend[s],
     * released by its st.release) are visible without a separate MEMBAR */
    while (cas_acquire_gpu(&c->claim[s], 0u, 1u) != 0u) {
        __nanosleep(ns);
        if (ns < 1024) ns <<= 1;
        if (expired(c, t0)) { wd_log(c, s, 0u, nr, GSYS_WD_CLAIM); return NOSLOT; }
    }
    // A non-blocking caller hands the claim back at once but the host may still be serving its
    // request (P24.34: the CPU sets the slot free): reuse waits for that completion word.
    const unsigned pend = c->nbpend[s];
    if (pend) {
        t0 = 0ull;
        while ((unsigned)(ld_relaxed_sys(c->hdone + s) >> 32) != pend) {
            __nanosleep(c->poll_ns_host);
            // the slot stays claimed (poisoned) until gsys_wait has drained the service
            if (expired(c, t0)) { wd_log(c, s, pend, nr, GSYS_WD_NBPEND); return NOSLOT; }
        }
        fence_acq_rel_sys();
        c->nbpend[s] = 0u;
        // reading B15: a small deferred pull of that request nobody consumed yet lands now, before
        // this caller's request can overtake it -- so at most one small pull per slot stays pending
        if (c->nbrec) consume_small_deferred(c, c->nbpos[s]);
    }
    return s;
}

/* ------------------------------------------------------------------ a3: marshal
 * args[0..5] as three 128-bit stores, then {nr, flags, seq, state=READY} as the fourth 128-bit
 * store of the 64 B line (P24.12: "populates the slot ... and changes the state to ready";
 * P24.13: the blocking bit travels in flags).  Returns the request's sequence number. */
__device__ __forceinline__ unsigned marshal(const gsys_dev_ctx* c, unsigned s, unsigned nr, unsigned flags,
                                            const unsigned long long a[6]) {
    unsigned seq = c->seqs[s] + 1u;
    if (seq == 0u) seq = 1u;
    c->seqs[s] = seq;
    trace(c, s, seq, GSYS_FREE, GSYS_POPULATING, !(flags & GSYS_NONBLOCKING), nr);
    uint4* line = reinterpret_cast<uint4*>(c->area + s);
    st_v4_sys(line + 0, make_uint4((unsigned)a[0], (unsigned)(a[0] >> 32), (unsigned)a[1], (unsigned)(a[1] >> 32)));
    st_v4_sys(line + 1, make_uint4((unsigned)a[2], (unsigned)(a[2] >> 32), (unsigned)a[3], (unsigned)(a[3] >> 32)));
    st_v4_sys(line + 2, make_uint4((unsigned)a[4], (unsigned)(a[4] >> 32), (unsigned)a[5], (unsigned)(a[5] >> 32)));
    st_v4_sys(line + 3, make_uint4(nr, flags, seq, (unsigned)GSYS_READY));
    trace(c, s, seq, GSYS_POPULATING, GSYS_READY, !(flags & GSYS_NONBLOCKING), nr);
    return seq;
}

/* ------------------------------------------------------------------ a4: publish + doorbell
 * __threadfence_system() orders the slot line before the doorbell entry; the entry position is
 * taken with one warp-aggregated atomicAdd for all lanes of the warp calling together (the
 * "scalar wavefront instruction" of P24.14).  Entry = (position+1) << 32 | slot, so the host
 * recognises a fresh entry without the ring ever being cleared. */
__device__ __forceinline__ unsigned doorbell(const gsys_dev_ctx* c, unsigned s) {
#if defined(GSYS_DOORBELL_SC)
    __threadfence_system();
#else
    fence_acq_rel_sys();   /* release: the slot line (and inline input) before the entry */
#endif
    unsigned mask = __activemask();
    unsigned lane = laneid();
    unsigned leader = __ffs(mask) - 1u;
    unsigned base = 0;
    if (lane == leader) base = atomicAdd(c->ring_tail, (unsigned)__popc(mask));
    base = __shfl_sync(mask, base, leader);
    unsigned pos = base + (unsigned)__popc(mask & lanemask_lt());
    st_relaxed_sys(c->ring + (pos & c->ring_mask), ((unsigned long long)(pos + 1u) << 32) | s);
    return pos;
}

/* ------------------------------------------------------------------ a5: completion
 * Blocking callers poll the slot's completion word until it carries their sequence number:
 * the device-memory word (L2-resident; written by a stream memory operation after the DMA) or,
 * for GSYS_HOSTBUF / inline / pulled calls, the host-mapped word the service stores directly
 * (each poll is one PCIe read, so the caller first sleeps a learned hint).  false: the watchdog
 * expired (logged; the slot stays claimed). */
__device__ __forceinline__ bool wait_done(const gsys_dev_ctx* c, unsigned s, unsigned seq, bool host, bool nohint,
                                          unsigned nr, long long& ret) {
    unsigned long long v;
    unsigned long long t0 = 0ull;
    if (!host) {
        const unsigned long long* m = c->mirror + s;
        unsigned ns = 64;
        for (;;) {
            v = GSYS_POLL_LOAD(m);
            if ((unsigned)(v >> 32) == seq) break;
            __nanosleep(ns);
            ns = ns < c->poll_ns_max ? ns << 1 : c->poll_ns_max;
            if (expired(c, t0)) { wd_log(c, s, seq, nr, GSYS_WD_COMPLETION); return false; }
        }
    } else {
        // every poll is a PCIe round trip, so a waiting caller first sleeps for the slot's learned
        // "sleep hint" and then polls at a fixed (short) interval.  The hint adapts on how the
        // wait went: answered by the first poll means it may have overslept (shrink by 1/4); more
        // than 2 polls means it woke too early (grow by half the time spent polling, measured on
        // %globaltimer), so the sleep converges just below the service latency without feeding on
        // its own length, whatever the poll interval.
        const unsigned long long* m = c->hdone + s;
        nohint = nohint || c->no_hint;
        const unsigned hint = nohint ? 0u : c->lat_hint[s];
        unsigned left = hint;
        while (left > 0) {
            const unsigned d = left > 100000u ? 100000u : left;
            __nanosleep(d);
            left -= d;
        }
        unsigned polls = 0;
        const unsigned long long tp = globaltimer();
        if (c->diag) { atomicAdd(c->diag + 5, (unsigned long long)hint); }
        for (;;) {
            v = GSYS_POLL_LOAD(m);
            polls++;
            if ((unsigned)(v >> 32) == seq) break;
            __nanosleep(c->poll_ns_host);
            if (expired(c, t0)) { wd_log(c, s, seq, nr, GSYS_WD_COMPLETION); return false; }
        }
        if (c->diag) atomicAdd(c->diag + 6, (unsigned long long)polls);
        if (!nohint) {
            unsigned long long nh = hint;
            if (polls <= 1) nh = hint - (hint >> 2);
            else if (polls > 2) nh = hint + ((globaltimer() - tp) >> 1);
            c->lat_hint[s] = nh > 200000ull ? 200000u : (unsigned)nh;
        }
    }
#ifdef GSYS_POLL_RELAXED_FENCE
    fence_acq_rel_sys();   /* diagnostic variant: relaxed polls + one fence (round-1 original) */
#endif
    /* the polls are acquire loads: the payload (device memory after the DMA, or the inline / pull
     * area the host wrote before its release store) is read after the completion word, with no
     * separate system-scope fence (a MEMBAR.SYS per call) */
    ret = (long long)(int)(unsigned)(v & 0xffffffffull);
    return true;
}

/* "The work-item can consume the result and continue execution" (P24.36; reading A3): the caller
 * returns the slot to free -- the host-visible state word of the line (a posted store) and the
 * device claim word.  release(): after the caller read host-written data (inline result, pull
 * area) -- the acquire/release pair orders those loads before the next owner's claim; with
 * `bounce`, the state store is a system-scope release, because the host recycles the bounce range
 * the work-group just copied from as soon as it sees the slot free. */
__device__ __forceinline__ void set_state_free(const gsys_dev_ctx* c, unsigned s, bool sys_release) {
    unsigned* st = &c->area[s].state;
    if (sys_release) asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(st), "r"((unsigned)GSYS_FREE) : "memory");
    else asm volatile("st.relaxed.sys.global.u32 [%0], %1;" :: "l"(st), "r"((unsigned)GSYS_FREE) : "memory");
}
__device__ __forceinline__ void release(const gsys_dev_ctx* c, unsigned s, unsigned seq, unsigned nr,
                                        bool bounce = false) {
    trace(c, s, seq, GSYS_FINISHED, GSYS_FREE, true, nr);
    set_state_free(c, s, bounce);
    st_release_gpu(&c->claim[s], 0u);
}
/* Release of a blocking call that read nothing host-written after its completion: the only data
 * the slot's next owner needs (seqs[s]) was ordered by the doorbell's fence.acq_rel.sys, and the
 * acquire poll keeps this store after the completion, so fence + relaxed store is the release
 * pattern already -- no second MEMBAR. */
__device__ __forceinline__ void release_after_fence(const gsys_dev_ctx* c, unsigned s, unsigned seq, unsigned nr) {
    trace(c, s, seq, GSYS_FINISHED, GSYS_FREE, true, nr);
    set_state_free(c, s, false);
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" :: "l"(&c->claim[s]), "r"(0u) : "memory");
}

/* ------------------------------------------------------------------ pull (reading B12)
 * A blocking pread into memory the host cannot write cheaply (device memory) is served into a
 * host-mapped area owned by the slot, completed with a host store, and copied to the destination
 * by the GPU (SM reads over PCIe) -- no copy-engine transfer and no stream memory operation,
 * whose fixed costs dominate small reads.  The area is the slot's inline line for n <= 256 B,
 * or, for a work-group's caller (cooperative copy) in a slot with s % 32 == 0, the slot's
 * pull_big_bytes area.  The slot stays claimed until the copy is done, so the host never
 * refills an area that is still being read.  Larger work-group reads (ctx->pull_bounce) land in
 * the serving worker's host-mapped bounce ring; the host passes the range's device address back
 * in args[1] (the argument field "re-purposed for the return value", P24.9) and recycles the
 * range once the work-group has set the slot free. */
__device__ __forceinline__ const unsigned char* pull_src(const gsys_dev_ctx* c, unsigned s, unsigned long long n,
                                                         bool coop) {
    if (n == 0ull) return nullptr;
    if (n <= GSYS_INLINE_BYTES) return c->inline_buf + (size_t)s * GSYS_INLINE_BYTES;
    if (coop && (s & 31u) == 0u && n <= c->pull_big_bytes) return c->pull_big + (size_t)(s >> 5) * c->pull_big_bytes;
    return nullptr;
}

/* 16 bytes v to d (any alignment), at most `left` of them */
__device__ __forceinline__ void store16(unsigned char* d, const uint4& v, long long left) {
    const uintptr_t da = (uintptr_t)d;
    if (left >= 16 && (da & 15u) == 0u) {
        *reinterpret_cast<uint4*>(d) = v;
    } else if (left >= 16 && (da & 3u) == 0u) {
        unsigned* d4 = reinterpret_cast<unsigned*>(d);
        d4[0] = v.x; d4[1] = v.y; d4[2] = v.z; d4[3] = v.w;
    } else {
        const unsigned m = left >= 16 ? 16u : (unsigned)left;
        for (unsigned b = 0; b < m; b++) {
            const unsigned w = b < 8u ? (b < 4u ? v.x : v.y) : (b < 12u ? v.z : v.w);
            d[b] = (unsigned char)(w >> (8u * (b & 3u)));
        }
    }
}

/* Copy r bytes of a pull area (16-byte aligned, host-mapped) to dst (any alignment); threads
 * tid = 0..nt-1 share the work, four pipelined loads at a time per thread (ld_v4_after_acquire:
 * the caller acquired the completion word; the other threads follow it through Bar2). */
__device__ __forceinline__ void pull_copy(const unsigned char* src, unsigned char* dst, long long r, unsigned tid,
                                          unsigned nt) {
    const unsigned n16 = (unsigned)((r + 15) >> 4);
    const uint4* s4 = reinterpret_cast<const uint4*>(src);
    const uint4 z = make_uint4(0u, 0u, 0u, 0u);
    for (unsigned i = tid; i < n16; i += 4u * nt) {
        const unsigned i1 = i + nt, i2 = i + 2u * nt, i3 = i + 3u * nt;
        const uint4 v0 = ld_v4_after_acquire(s4 + i);
        const uint4 v1 = i1 < n16 ? ld_v4_after_acquire(s4 + i1) : z;
        const uint4 v2 = i2 < n16 ? ld_v4_after_acquire(s4 + i2) : z;
        const uint4 v3 = i3 < n16 ? ld_v4_after_acquire(s4 + i3) : z;
        store16(dst + 16u * i, v0, r - 16ll * i);
        if (i1 < n16) store16(dst + 16u * i1, v1, r - 16ll * i1);
        if (i2 < n16) store16(dst + 16u * i2, v2, r - 16ll * i2);
        if (i3 < n16) store16(dst + 16u * i3, v3, r - 16ll * i3);
    }
}

/* One thread copies r bytes of a host-mapped area (16-byte aligned) to dst: eight 16-byte loads in
 * flight per round trip over PCIe. */
__device__ __forceinline__ void pull_copy_thread(const unsigned char* src, unsigned char* dst, long long r) {
    const unsigned n16 = (unsigned)((r + 15) >> 4);
    const uint4* s4 = reinterpret_cast<const uint4*>(src);
    for (unsigned i = 0; i < n16; i += 8u) {
        uint4 v[8];
#pragma unroll
        for (unsigned k = 0; k < 8u; k++) v[k] = i + k < n16 ? ld_v4_after_acquire(s4 + i + k) : make_uint4(0u, 0u, 0u, 0u);
#pragma unroll
        for (unsigned k = 0; k < 8u; k++)
            if (i + k < n16) store16(dst + 16u * (i + k), v[k], r - 16ll * (i + k));
    }
}

/* Copy a deferred pull (threads tid = 0..nt-1 of the caller's scope), then mark it consumed. */
__device__ __forceinline__ void finish_deferred(const gsys_nbrec* q, unsigned tid, unsigned nt) {
    const uint4 h = ld_v4_after_acquire(reinterpret_cast<const uint4*>(q));
    const uint4 t = ld_v4_after_acquire(reinterpret_cast<const uint4*>(q) + 1);
    const unsigned char* src = reinterpret_cast<const unsigned char*>((unsigned long long)h.x |
                                                                      ((unsigned long long)h.y << 32));
    unsigned char* dst = reinterpret_cast<unsigned char*>((unsigned long long)h.z | ((unsigned long long)h.w << 32));
    const long long r = (long long)((unsigned long long)t.x | ((unsigned long long)t.y << 32));
    if (nt == 1u) pull_copy_thread(src, dst, r);
    else pull_copy(src, dst, r, tid, nt);
}
__device__ __forceinline__ void mark_consumed(const gsys_nbrec* q) {
    unsigned* cons = const_cast<unsigned*>(&q->consumed);
    asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(cons), "r"(1u) : "memory");
}

/* A pull the caller's scope finishes (work-group cooperative copy): filled by call_thread. */
struct PullOut {
    const unsigned char* src = nullptr;
    unsigned slot = 0, seq = 0, nr = 0;
    bool bounce = false;
};

/* One thread, one request: claim -> (inline input) -> marshal -> publish -> (poll).  A non-blocking
 * request's slot is reused only after the host has served it (P24.34, A15); `tok` (may be null)
 * receives its (slot, seq) for gsys_wait_token().  io.out: for GSYS_F_INLINE calls, where the
 * host's inline result is copied after completion.  po: when set (a work-group caller), a pulled
 * pread's copy and the slot's release are left to the caller's scope; otherwise this thread
 * copies (inline-size pulls only). */
__device__ __forceinline__ long long call_thread(const gsys_dev_ctx* c, unsigned nr, unsigned flags,
                                                 const unsigned long long a[6], const InlineIO& io = InlineIO(),
                                                 PullOut* po = nullptr, gsys_token* tok = nullptr) {
    const bool blocking = !(flags & GSYS_NONBLOCKING);
    const unsigned long long d0 = c->diag ? globaltimer() : 0ull;
    unsigned s = claim(c, nr);
    if (s == NOSLOT) {
        if (tok) { tok->slot = 0u; tok->seq = 0u; }
        return -ETIMEDOUT;
    }
    const unsigned long long d1 = c->diag ? globaltimer() : 0ull;
    const unsigned char* psrc = nullptr;
    // non-blocking pread into device memory: served into a host-mapped range and pulled later (B15)
    // (work-item and work-group callers; a kernel-scope call is one thread the whole grid waits on:
    // it keeps the copy engine)
    const unsigned gran = flags & GSYS_GRAN_MASK;
    if (nr == GSYS_NR_PREAD64 && !blocking && !(flags & GSYS_HOSTBUF) && c->nbrec != nullptr && a[2] > 0ull &&
        gran != GSYS_KERNEL)
        flags |= GSYS_F_DEFER;
    if (nr == GSYS_NR_PREAD64 && blocking && !(flags & GSYS_HOSTBUF)) {
        psrc = pull_src(c, s, a[2], po != nullptr);
        if (psrc) flags |= GSYS_F_PULL;
        // bounce pull (B13): a work-group copies cooperatively; work-item callers copy with their
        // converged warp (or alone), which pays only up to 64 KiB; a kernel-scope call is copied by
        // the calling block, up to 1 MiB (larger reads keep the DMA path)
        else if (c->pull_bounce && a[2] > 0ull &&
                 ((po != nullptr && gran == GSYS_WG) || (gran == GSYS_WI && a[2] <= (64ull << 10)) ||
                  (po != nullptr && gran == GSYS_KERNEL && a[2] <= (1ull << 20))))
            flags |= GSYS_F_PULLB;
    }
    if (io.in != nullptr) {   /* input payload into the inline line; published by marshal's fence */
        uint4* dst = reinterpret_cast<uint4*>(c->inline_buf + (size_t)s * GSYS_INLINE_BYTES);
        const unsigned char* src = reinterpret_cast<const unsigned char*>(io.in);
        for (unsigned i = 0; i < (io.in_bytes + 15u) / 16u; i++) {
            uint4 v;
            unsigned char* vb = reinterpret_cast<unsigned char*>(&v);
            for (unsigned k = 0; k < 16u; k++) vb[k] = 16u * i + k < io.in_bytes ? src[16u * i + k] : 0u;
            st_v4_sys(dst + i, v);
        }
        flags |= GSYS_F_INLINE_IN;
    }
    unsigned seq = marshal(c, s, nr, flags, a);
    const unsigned pos = doorbell(c, s);
    if (!blocking) {
        c->nbpend[s] = seq;
        c->nbpos[s] = pos;
        if (tok) { tok->slot = s; tok->seq = seq; tok->pos = pos; }
        st_release_gpu(&c->claim[s], 0u);
        return 0;
    }
    const unsigned long long d2 = c->diag ? globaltimer() : 0ull;
    long long r = 0;
    if (!wait_done(c, s, seq,
                   !c->memop_completion || (flags & (GSYS_HOSTBUF | GSYS_F_INLINE | GSYS_F_PULL | GSYS_F_PULLB)) != 0u,
                   (flags & GSYS_F_NOHINT) != 0u, nr, r))
        return -ETIMEDOUT;   /* slot left claimed: the host may still complete into it */
    if (c->diag) {   /* phase diagnostics: claim, marshal+publish, wait, (copy+release below) */
        const unsigned long long d3 = globaltimer();
        atomicAdd(c->diag + 0, d1 - d0);
        atomicAdd(c->diag + 1, d2 - d1);
        atomicAdd(c->diag + 2, d3 - d2);
        atomicAdd(c->diag + 4, 1ull);
        atomicAdd(c->diag + 7, (unsigned long long)-(long long)d3);   /* + end time below */
    }
    if (flags & GSYS_F_PULLB) {   /* copy from the worker's bounce (the work-group, or this thread), then release */
        const uint4 a01 = ld_v4_after_acquire(reinterpret_cast<const uint4*>(c->area + s));   /* args[1] = source */
        const unsigned char* src =
            r > 0 ? reinterpret_cast<const unsigned char*>((uintptr_t)a01.z | ((uintptr_t)a01.w << 32)) : nullptr;
        if (po != nullptr) {
            po->src = src; po->slot = s; po->seq = seq; po->nr = nr; po->bounce = true;
            if (c->diag) atomicAdd(c->diag + 7, globaltimer());
            return r;
        }
        if (src != nullptr) pull_copy_thread(src, reinterpret_cast<unsigned char*>(a[1]), r);
        release(c, s, seq, nr, true);
        if (c->diag) atomicAdd(c->diag + 7, globaltimer());
        return r;
    }
    if (psrc != nullptr && r > 0) {
        if (po != nullptr) {   /* the work-group copies and releases (wg_call) */
            po->src = psrc; po->slot = s; po->seq = seq; po->nr = nr; po->bounce = false;
            if (c->diag) atomicAdd(c->diag + 7, globaltimer());
            return r;
        }
        pull_copy(psrc, reinterpret_cast<unsigned char*>(a[1]), r, 0u, 1u);
    }
    if (io.out != nullptr && r >= 0) {
        const uint4* src = reinterpret_cast<const uint4*>(c->inline_buf + (size_t)s * GSYS_INLINE_BYTES);
        uint4* dst = reinterpret_cast<uint4*>(io.out);
        // every piece's load is issued before the first store: one PCIe round trip for the result
        const unsigned n16 = io.out_bytes / 16u;
        uint4 t[GSYS_INLINE_BYTES / 16];
#pragma unroll
        for (unsigned i = 0; i < GSYS_INLINE_BYTES / 16; i++)
            if (i < n16) t[i] = ld_v4_after_acquire(src + i);
#pragma unroll
        for (unsigned i = 0; i < GSYS_INLINE_BYTES / 16; i++)
            if (i < n16) dst[i] = t[i];
    }
    if (io.out != nullptr || psrc != nullptr) release(c, s, seq, nr);
    else release_after_fence(c, s, seq, nr);
    if (c->diag) atomicAdd(c->diag + 7, globaltimer());
    return r;
}

/* ------------------------------------------------------------------ a1/a6: granularity + ordering
 * Work-group (PAPER.md:22 P22.40-42): thread 0 is the designated caller; strong = barrier
 * before and after; relaxed keeps the barrier before for consumer calls, after for producer
 * calls.  The result reaches every thread through a shared-memory double buffer whose parity is
 * broadcast by the Bar2 barrier itself (__syncthreads_or), so back-to-back calls never race.
 * Relaxed consumer (Bar2 removed): the caller's warp waits with it and gets the result, the
 * other warps proceed at once and get 0 (reading A17, P28.3). */
__device__ __forceinline__ long long wg_call(const gsys_dev_ctx* c, unsigned nr, unsigned flags, bool producer,
                                             const unsigned long long a[6], const InlineIO& io = InlineIO(),
                                             gsys_token* tok = nullptr) {
    __shared__ long long s_ret[2];
    __shared__ unsigned s_par;
    __shared__ const unsigned char* s_psrc[2];
    __shared__ unsigned char* s_pdst[2];
    __shared__ unsigned s_prel[2];
    const bool strong = !(flags & GSYS_RELAXED);
    const bool bar1 = strong || !producer;
    const bool bar2 = strong || producer;
    const unsigned tid = block_tid();
    if (bar1) {
        // Bar1 doubles as the broadcast of a small deferred pull (B15) still pending on the
        // caller's slot: the whole work-group copies it instead of the caller alone in claim()
        __shared__ const gsys_nbrec* s_dq;
        int pend = 0;
        if (tid == 0 && c->nbrec) {
            s_dq = small_deferred_pending(c, hw_slot(c));
            pend = s_dq != nullptr;
        }
        if (__syncthreads_or(pend)) {
            finish_deferred(s_dq, tid, block_threads());
            __syncthreads();
            if (tid == 0) mark_consumed(s_dq);
        }
    } else if (c->nbrec && tid < 32u && nr == GSYS_NR_PREAD64 && !(flags & GSYS_HOSTBUF)) {
        // relaxed producer (no barrier before the call): warp 0 -- converged here, every thread of
        // the work-group makes the call -- lands such a pull instead of the caller alone in claim()
        const unsigned nt = block_threads();
        const unsigned wm = nt >= 32u ? 0xffffffffu : ((1u << nt) - 1u);
        const gsys_nbrec* q = tid == 0 ? small_deferred_pending(c, hw_slot(c)) : nullptr;
        q = reinterpret_cast<const gsys_nbrec*>(__shfl_sync(wm, (unsigned long long)q, 0));
        if (q) {
            __syncwarp(wm);
            finish_deferred(q, tid, __popc(wm));
            __syncwarp(wm);
            if (tid == 0) mark_consumed(q);
        }
    }
    long long r = 0;
    PullOut po;
    if (tid == 0)
        r = call_thread(c, nr, flags | (producer ? GSYS_F_PRODUCER : 0u), a, io, bar2 ? &po : nullptr, tok);
    if (bar2) {
        unsigned p = 0;
        if (tid == 0) {
            p = (s_par ^ 1u) & 1u; s_par = p; s_ret[p] = r;
            s_psrc[p] = po.src; s_pdst[p] = reinterpret_cast<unsigned char*>(a[1]);
            s_prel[p] = (po.src != nullptr || po.bounce) ? 1u : 0u;
        }
        p = (unsigned)__syncthreads_or(tid == 0 ? (int)p : 0);
        const long long rv = s_ret[p];
        const unsigned char* src = s_psrc[p];
        if (src != nullptr && rv > 0) {   /* pulled pread (reading B12): the whole work-group copies */
            pull_copy(src, s_pdst[p], rv, tid, block_threads());
        }
        if (s_prel[p]) {   /* the work-group's copy is done: thread 0 returns the slot */
            __syncthreads();
            if (tid == 0) release(c, po.slot, po.seq, po.nr, po.bounce);
        }
        return rv;
    }
    if (tid < 32) {
        unsigned nt = block_threads();
        unsigned m = nt >= 32 ? 0xffffffffu : ((1u << nt) - 1u);
        r = __shfl_sync(m, r, 0);
        return r;
    }
    return 0;
}

/* Work-item (P20.31 "work-item invocations imply strong ordering"): every calling lane issues
 * its own request; the claim spins diverge, publication and the doorbell are warp-aggregated.
 * Device-buffer preads are copied by the lanes of the warp that reach the call together:
 * blocking ones are pulled (B12, B13) and the lanes copy every payload together -- 16-byte pieces
 * spread over the lanes, one PCIe round trip per 512 B instead of a lone thread's loop -- before
 * each returns its own slot; for non-blocking ones the lanes land the small deferred pulls (B15)
 * their slots still hold, together, before claiming. */
__device__ __forceinline__ long long wi_call(const gsys_dev_ctx* c, unsigned nr, unsigned flags, bool producer,
                                             const unsigned long long a[6], const InlineIO& io = InlineIO(),
                                             gsys_token* tok = nullptr) {
    const unsigned f = (flags & ~GSYS_RELAXED) | (producer ? GSYS_F_PRODUCER : 0u);
    const bool coop = nr == GSYS_NR_PREAD64 && !(flags & (GSYS_NONBLOCKING | GSYS_HOSTBUF));
    const bool nbdev = nr == GSYS_NR_PREAD64 && (flags & GSYS_NONBLOCKING) && !(flags & GSYS_HOSTBUF) &&
                       c->nbrec != nullptr;
    const unsigned am = __activemask();
    const unsigned m = __ballot_sync(am, coop);
    const unsigned mnb = __ballot_sync(am, nbdev);
    if (nbdev) {
        // a small deferred pull (B15) still pending on a lane's slot is copied by the converged
        // lanes together before the claims, instead of by its lane alone inside claim()
        const gsys_nbrec* q = small_deferred_pending(c, hw_slot(c));
        __syncwarp(mnb);   /* each lane's acquire of its record before the others read its bytes */
        unsigned todo = __ballot_sync(mnb, q != nullptr);
        const unsigned rank = __popc(mnb & lanemask_lt()), nt = __popc(mnb);
        while (todo) {
            const int k = __ffs(todo) - 1;
            todo &= todo - 1u;
            finish_deferred(reinterpret_cast<const gsys_nbrec*>(__shfl_sync(mnb, (unsigned long long)q, k)), rank, nt);
        }
        __syncwarp(mnb);
        if (q) mark_consumed(q);
    }
    if (!coop) return call_thread(c, nr, f, a, io, nullptr, tok);
    PullOut po;
    const long long r = call_thread(c, nr, f, a, io, &po, tok);
    __syncwarp(m);   /* every lane's completion acquired before any lane reads another's payload */
    unsigned todo = __ballot_sync(m, po.src != nullptr && r > 0);
    const unsigned rank = __popc(m & lanemask_lt()), nt = __popc(m);
    while (todo) {
        const int k = __ffs(todo) - 1;
        todo &= todo - 1u;
        const unsigned char* src =
            reinterpret_cast<const unsigned char*>(__shfl_sync(m, (unsigned long long)po.src, k));
        unsigned char* dst = reinterpret_cast<unsigned char*>(__shfl_sync(m, a[1], k));
        const long long n = __shfl_sync(m, r, k);
        pull_copy(src, dst, n, rank, nt);
    }
    __syncwarp(m);   /* the copies are done: the slots (and their bounce ranges) can be returned */
    if (po.src != nullptr || po.bounce) release(c, po.slot, po.seq, po.nr, po.bounce);
    return r;
}

/* Kernel (P20.16-21, P20.33): relaxed only, -EINVAL for strong (reading A13).  Per call site and
 * per round (the block's n-th call at that site) a record in device memory counts arrivals.
 * Producer: the FIRST block to arrive calls (it is resident by definition, so nobody can wait
 * on a block that was never scheduled) and the others wait for its result -- the kernel-scope
 * "barrier after".  Consumer: the LAST block to arrive calls after every block published its
 * data (the "barrier before"), and nobody waits.  Both are deadlock-free for grids larger than
 * the co-resident capacity.  Sites are GSYS_SITE(0..GSYS_KSITES-1); another site is -EINVAL. */
__device__ __forceinline__ long long kernel_call(const gsys_dev_ctx* c, unsigned nr, unsigned flags, bool producer,
                                                 const unsigned long long a[6], const InlineIO& io = InlineIO()) {
    __shared__ long long s_kret[2];
    __shared__ unsigned s_kpar;
    __shared__ const unsigned char* s_ksrc;
    __shared__ unsigned s_kslot, s_kseq, s_knr, s_kbounce;
    __shared__ unsigned char* s_kdst;
    __shared__ gsys_kround* s_kround;
    __shared__ long long s_kpo_ret;
    int kcopy = 0;
    if (!(flags & GSYS_RELAXED)) return -EINVAL;
    const unsigned site = (flags >> 24) & 63u;
    if (site >= GSYS_KSITES) return -EINVAL;
    const unsigned tid = block_tid();
    const unsigned nb = gridDim.x * gridDim.y * gridDim.z;
    const unsigned bid = block_linear();
    if (!producer) __syncthreads();     /* block-level part of the barrier before */
    long long r = 0;
    if (tid == 0) {
        if (bid >= c->kblock_cap) {
            r = -ENOSPC;
        } else {
            unsigned* kb = c->kblock + (size_t)bid * GSYS_KSITES + site;
            unsigned round = *kb;
            *kb = round + 1u;
            if (round >= GSYS_KROUNDS) {
                r = -ENOSPC;
            } else {
                gsys_kround* k = c->krounds + (size_t)site * GSYS_KROUNDS + round;
                if (producer) {
                    unsigned t = atomicAdd(&k->arrive, 1u);
                    if (t == 0u) {
                        PullOut po;
                        r = call_thread(c, nr, flags | GSYS_F_PRODUCER, a, io, &po);
                        if (po.src != nullptr || po.bounce) {   /* pulled: the block copies, then publishes */
                            s_ksrc = po.src; s_kslot = po.slot; s_kseq = po.seq; s_knr = po.nr;
                            s_kbounce = po.bounce ? 1u : 0u;
                            s_kdst = reinterpret_cast<unsigned char*>(a[1]);
                            s_kround = k;
                            kcopy = 1;
                        } else {
                            k->ret = r;
                            __threadfence();
                            st_release_gpu(&k->done, 1u);
                        }
                    } else {
                        unsigned ns = 64;
                        unsigned long long t0 = 0ull;
                        bool ok = true;
                        while (ld_acquire_gpu(&k->done) == 0u) {
                            __nanosleep(ns);
                            if (ns < 2048) ns <<= 1;
                            if (expired(c, t0)) { wd_log(c, site, round, nr, GSYS_WD_KERNEL); ok = false; break; }
                        }
                        r = ok ? *(volatile long long*)&k->ret : -ETIMEDOUT;
                    }
                } else {
                    __threadfence();
                    unsigned t = atomicAdd(&k->arrive, 1u);
                    if (t == nb - 1u) {
                        __threadfence();
                        r = call_thread(c, nr, flags, a, io);
                    }
                }
            }
        }
    }
    if (producer) {
        if (__syncthreads_or(kcopy)) {   /* the first arriver's pulled pread: the whole block copies */
            if (tid == 0) s_kpo_ret = r;
            __syncthreads();
            const long long rv = s_kpo_ret;
            if (s_ksrc != nullptr && rv > 0) pull_copy(s_ksrc, s_kdst, rv, tid, block_threads());
            __syncthreads();
            if (tid == 0) {
                release(c, s_kslot, s_kseq, s_knr, s_kbounce != 0u);
                s_kround->ret = r;
                __threadfence();
                st_release_gpu(&s_kround->done, 1u);
            }
        }
        unsigned p = 0;
        if (tid == 0) { p = (s_kpar ^ 1u) & 1u; s_kpar = p; s_kret[p] = r; }
        p = (unsigned)__syncthreads_or(tid == 0 ? (int)p : 0);
        return s_kret[p];
    }
    return tid == 0 ? r : 0;
}

__device__ __forceinline__ bool flags_valid(unsigned flags) {
    unsigned g = flags & GSYS_GRAN_MASK;
    return g == GSYS_WI || g == GSYS_WG || g == GSYS_KERNEL;
}

/* Dispatch on granularity.  Invalid granularity -> -EINVAL (uniform across the scope). */
__device__ __forceinline__ long long invoke(const gsys_dev_ctx* c, unsigned nr, unsigned flags, bool producer,
                                            const unsigned long long a[6], const InlineIO& io = InlineIO(),
                                            gsys_token* tok = nullptr) {
    switch (flags & GSYS_GRAN_MASK) {
        case GSYS_WI: return wi_call(c, nr, flags, producer, a, io, tok);
        case GSYS_WG: return wg_call(c, nr, flags, producer, a, io, tok);
        case GSYS_KERNEL: return kernel_call(c, nr, flags, producer, a, io);
        default: return -EINVAL;
    }
}

/* Wait for the non-blocking request of `tok` (one thread's token) to complete: returns its result
 * if the slot's completion word still carries it, 0 if a later request on the slot completed
 * since (completions on a slot are in order, A15: ours is done, its result was overwritten --
 * errors still reach gsys_wait, reading A4), -ETIMEDOUT from the watchdog.  *rec receives the
 * request's deferred-pull record when it has bytes still to copy (B15), else nullptr. */
__device__ __forceinline__ long long wait_token_thread(const gsys_dev_ctx* c, const gsys_token& tok,
                                                       const gsys_nbrec** rec = nullptr) {
    if (rec) *rec = nullptr;
    if (tok.seq == 0u) return 0;
    const unsigned long long* m = c->hdone + tok.slot;
    unsigned long long t0 = 0ull;
    long long r = 0;
    for (;;) {
        const unsigned long long v = ld_acquire_sys(m);
        const unsigned got = (unsigned)(v >> 32);
        if (got == tok.seq) { r = (long long)(int)(unsigned)(v & 0xffffffffull); break; }
        if ((int)(got - tok.seq) > 0) break;
        __nanosleep(c->poll_ns_host);
        if (expired(c, t0)) { wd_log(c, tok.slot, tok.seq, 0u, GSYS_WD_TOKEN); return -ETIMEDOUT; }
    }
    if (rec && c->nbrec) {
        // the record is written before the completion word (acquired above)
        const gsys_nbrec* q = c->nbrec + (tok.pos & c->ring_mask);
        const uint4 t = ld_v4_after_acquire(reinterpret_cast<const uint4*>(q) + 1);   /* {ret, tag, consumed} */
        const uint4 h = ld_v4_after_acquire(reinterpret_cast<const uint4*>(q));       /* {src, dst}           */
        if (t.z == tok.pos + 1u && t.w == 0u && (h.x | h.y) != 0u && (long long)((unsigned long long)t.x |
                                                                                 ((unsigned long long)t.y << 32)) > 0) {
            if (claim_record(c, tok.pos)) *rec = q;    /* this waiter's scope copies it */
            else wait_consumed(c, q);                  /* another copier has it: wait for the bytes */
        }
    }
    return r;
}

}  // namespace gsys

/* ------------------------------------------------------------------ POSIX-shaped wrappers
 * Signatures follow POSIX plus the trailing GENESYS flags (P20.31-33).  Blocking calls return the
 * raw-syscall convention (>= 0, or -errno); non-blocking calls return 0 once published and report
 * errors at gsys_wait() (reading A4).  Producer (read-like) vs consumer (write-like) class per
 * P20.24-29; madvise and rt_sigqueueinfo are consumers (reading A7). */
__device__ __forceinline__ long long gsys_pread(const gsys_dev_ctx* c, int fd, void* buf, size_t n, long long off,
                                                unsigned gflags, gsys_token* tok = nullptr) {
    unsigned long long a[6] = {(unsigned long long)(long long)fd, (unsigned long long)buf, (unsigned long long)n,
                               (unsigned long long)off, 0ull, 0ull};
    return gsys::invoke(c, GSYS_NR_PREAD64, gflags, true, a, gsys::InlineIO(), tok);
}
/* Completion wait on an explicit token (the trailing `tok` of a non-blocking gsys_pread / pwrite /
 * sendto: for WG calls it must be visible to the whole work-group, e.g. __shared__; thread 0
 * writes it).  gflags' granularity
 * gives the scope: GSYS_WI -- the calling thread waits on its own token; GSYS_WG -- thread 0
 * waits on *tok and every thread of the block gets the result after a barrier (all must call).
 * GSYS_KERNEL: -EINVAL (the token lives in one block). */
__device__ __forceinline__ long long gsys_wait_token(const gsys_dev_ctx* c, const gsys_token* tok, unsigned gflags) {
    const unsigned g = gflags & GSYS_GRAN_MASK;
    if (g == GSYS_WI) {
        const gsys_nbrec* q = nullptr;
        const long long r = gsys::wait_token_thread(c, *tok, &q);
        if (q) { gsys::finish_deferred(q, 0u, 1u); gsys::mark_consumed(q); }
        return r;
    }
    if (g != GSYS_WG) return -EINVAL;
    __shared__ long long s_tret;
    __shared__ const gsys_nbrec* s_trec;
    __syncthreads();
    if (gsys::block_tid() == 0) s_tret = gsys::wait_token_thread(c, *tok, &s_trec);
    __syncthreads();
    const long long r = s_tret;
    const gsys_nbrec* q = s_trec;
    if (q) {   /* the deferred pull (B15): the whole work-group copies, thread 0 marks it consumed */
        gsys::finish_deferred(q, gsys::block_tid(), gsys::block_threads());
        __syncthreads();
        if (gsys::block_tid() == 0) gsys::mark_consumed(q);
    }
    __syncthreads();
    return r;
}
__device__ __forceinline__ long long gsys_pwrite(const gsys_dev_ctx* c, int fd, const void* buf, size_t n,
                                                 long long off, unsigned gflags, gsys_token* tok = nullptr) {
    unsigned long long a[6] = {(unsigned long long)(long long)fd, (unsigned long long)buf, (unsigned long long)n,
                               (unsigned long long)off, 0ull, 0ull};
    return gsys::invoke(c, GSYS_NR_PWRITE64, gflags, false, a, gsys::InlineIO(), tok);
}
/* getrusage: blocking calls land the 144 B struct rusage in the slot's inline line and the
 * caller copies it to `ru` (any pointer the thread can write, including local memory);
 * non-blocking calls hand a global `ru` to the host, which writes it asynchronously -- for a
 * thread-local `ru` the non-blocking result is discarded, as for every non-blocking call (P24.34). */
__device__ __forceinline__ long long gsys_getrusage(const gsys_dev_ctx* c, int who, void* ru, unsigned gflags) {
    const bool blocking = !(gflags & GSYS_NONBLOCKING);
    const bool inl = ru != nullptr && (blocking || !__isGlobal(ru));
    unsigned long long a[6] = {(unsigned long long)(long long)who, (unsigned long long)ru, 0ull, 0ull, 0ull, 0ull};
    gsys::InlineIO io;
    io.out = blocking ? ru : nullptr;
    io.out_bytes = 144u;
    return gsys::invoke(c, GSYS_NR_GETRUSAGE, gflags | (inl ? GSYS_F_INLINE : 0u), true, a, io);
}
__device__ __forceinline__ long long gsys_madvise(const gsys_dev_ctx* c, void* addr, size_t len, int advice,
                                                  unsigned gflags) {
    unsigned long long a[6] = {(unsigned long long)addr, (unsigned long long)len, (unsigned long long)(long long)advice,
                               0ull, 0ull, 0ull};
    return gsys::invoke(c, GSYS_NR_MADVISE, gflags, false, a);
}
__device__ __forceinline__ long long gsys_sendto(const gsys_dev_ctx* c, int fd, const void* buf, size_t n, int flags,
                                                 const void* to, unsigned tolen, unsigned gflags,
                                                 gsys_token* tok = nullptr) {
    unsigned long long a[6] = {(unsigned long long)(long long)fd, (unsigned long long)buf, (unsigned long long)n,
                               (unsigned long long)(long long)flags, (unsigned long long)to, (unsigned long long)tolen};
    return gsys::invoke(c, GSYS_NR_SENDTO, gflags | GSYS_F_NOHINT, false, a, gsys::InlineIO(), tok);
}
__device__ __forceinline__ long long gsys_recvfrom(const gsys_dev_ctx* c, int fd, void* buf, size_t n, int flags,
                                                   void* from, unsigned* fromlen, unsigned gflags) {
    unsigned long long a[6] = {(unsigned long long)(long long)fd, (unsigned long long)buf, (unsigned long long)n,
                               (unsigned long long)(long long)flags, (unsigned long long)from,
                               (unsigned long long)fromlen};
    return gsys::invoke(c, GSYS_NR_RECVFROM, gflags | GSYS_F_NOHINT, true, a);
}
/* rt_sigqueueinfo: the 128 B siginfo travels in the slot's inline line (copied by the caller before
 * publishing), so `info` may live anywhere the caller can read -- registers/local memory included --
 * and a non-blocking call does not have to keep it alive. */
__device__ __forceinline__ long long gsys_rt_sigqueueinfo(const gsys_dev_ctx* c, int tgid, int sig, const void* info,
                                                          unsigned gflags) {
    unsigned long long a[6] = {(unsigned long long)(long long)tgid, (unsigned long long)(long long)sig,
                               (unsigned long long)info, 0ull, 0ull, 0ull};
    gsys::InlineIO io;
    io.in = info;
    io.in_bytes = info ? 128u : 0u;
    return gsys::invoke(c, GSYS_NR_RT_SIGQUEUEINFO, gflags, false, a, io);
}

#endif /* __CUDACC__ */
#endif /* GSYS_DEVICE_CUH */
