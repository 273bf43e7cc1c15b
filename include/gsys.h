/*
 * gsys.h -- C-ABI of libgsys: GPU-issued POSIX system calls on NVIDIA B200 (sm_100a).
 *
 * A from-scratch, B200-native take on GENESYS (Vesely et al., "Generic System Calls for GPUs",
 * ISCA 2018; /root/reference/PAPER.md).  GPU threads claim a slot of a shared "syscall area"
 * (sec. III step 1), publish the call and ring a doorbell (step 2, the paper's
 * s_sendmsg interrupt, PAPER.md:24 P24.14), a host service executes the real POSIX call
 * (steps 3-4, P24.16-21) and returns the result into the slot (step 5, P24.32-36).  The paper's
 * modified Linux kernel / interrupt path is replaced by a user-space service thread pool,
 * because the box's kernel cannot be changed (BASELINE.json north_star).
 *
 * Every entry point is `extern "C"`, takes plain pointers and sizes, and returns 0 (or a
 * documented non-negative value) on success and -errno on failure.  One instance exists per CUDA
 * device per process; it is bound to the device that is current when gsys_init() is called, and
 * every other entry point acts on the instance of the *current* device.
 *
 * Ownership: the library owns the syscall area, claim words, doorbell ring, bounce buffers,
 * service threads and their CUDA streams.  The caller owns file descriptors (they must stay open
 * until gsys_wait() returns for every launch that uses them), every buffer it passes (device
 * memory from cudaMalloc/PyTorch, or pinned host-mapped memory; they must stay alive until the
 * call completes -- for non-blocking calls until gsys_wait()), and the CUDA streams it passes.
 */
#ifndef GSYS_H
#define GSYS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---------------------------------------------------------------- slot layout (reading A1)
 * "64 bytes per slot ... the requested system call number, the request state, system call
 * arguments (as many as 6, in Linux), and padding to avoid false sharing.  The field for
 * arguments is also re-purposed for the return value" (sec. VI, P24.7-9).
 * One 64 B, 64 B-aligned line per slot; args[0] carries the i64 result back. */
typedef struct gsys_slot {
    uint64_t args[6];   /* bytes  0..47: syscall arguments; args[0] <- return value        */
    uint32_t nr;        /* bytes 48..51: Linux x86-64 syscall number (pread64 = 17, ...)    */
    uint32_t flags;     /* bytes 52..55: GSYS_* granularity/blocking/ordering bits (P24.13)  */
    uint32_t seq;       /* bytes 56..59: per-slot request sequence number                   */
    uint32_t state;     /* bytes 60..63: gsys_state                                         */
} gsys_slot;

/* Slot states (PAPER.md:24 P24.10-34, Fig. 6 caption PAPER.md:22; reading A2). */
enum gsys_state {
    GSYS_FREE = 0,        /* no request                                        */
    GSYS_POPULATING = 1,  /* claimed by a GPU thread (cmp-swap, P24.10, P24.46) */
    GSYS_READY = 2,       /* published, doorbell rung (P24.12-14)               */
    GSYS_PROCESSING = 3,  /* picked up by a host worker (P24.20)                */
    GSYS_FINISHED = 4     /* blocking call done, result in args[0] (P24.33)     */
};

/* ---------------------------------------------------------------- per-call flags
 * Granularity: exactly one of WI / WG / KERNEL (sec. V-A "work-item, work-group,
 * or kernel").  Blocking is the default (P20.34-46).  Ordering: strong is the default; relaxed
 * removes Bar1 for producer calls or Bar2 for consumer calls (PAPER.md:20 P20.24-29, PAPER.md:22
 * P22.41-42).  WI calls are always strong (P20.31); KERNEL calls must be relaxed (P20.33), so
 * KERNEL|STRONG returns -EINVAL. */
#define GSYS_WI          0x01u
#define GSYS_WG          0x02u
#define GSYS_KERNEL      0x04u
#define GSYS_GRAN_MASK   0x07u
#define GSYS_BLOCKING    0x00u
#define GSYS_NONBLOCKING 0x08u
#define GSYS_STRONG      0x00u
#define GSYS_RELAXED     0x10u
#define GSYS_WEAK        GSYS_RELAXED
#define GSYS_KSITES_MAX  8u
#define GSYS_SITE(k)     (((uint32_t)(k) & 63u) << 24)   /* kernel-scope call site 0..7; 8..63 -> -EINVAL */
/* Completion through system memory: the caller's buffer is pinned host-mapped memory, so the
 * host service performs the call in place and signals completion with a plain store into the
 * slot's host-mapped completion word, which the GPU polls over PCIe (the paper's "CPU-GPU
 * communication ... via atomic reads/writes in system memory", PAPER.md:16 P16.8).  Without
 * the flag the GPU polls a device-memory completion word written by a CUDA stream memory
 * operation ordered after the payload DMA.  Either way the result is correct for any buffer;
 * the flag picks the fast path. */
#define GSYS_HOSTBUF     0x20u
/* internal bits set by the device library in the slot's flags word */
#define GSYS_F_PRODUCER  0x100u   /* call class: producer (read-like), P20.24-29            */
#define GSYS_F_INLINE    0x200u   /* small result goes to the slot's inline payload line    */
#define GSYS_F_INLINE_IN 0x400u   /* small input (siginfo, sockaddr) is in the inline line   */
#define GSYS_F_NOHINT    0x800u   /* unpredictable latency (network): poll without the learned sleep */
#define GSYS_F_PULL      0x1000u  /* blocking pread: the host reads into the slot's host-mapped pull
                                     area and the GPU copies it to the destination (reading B12)  */
#define GSYS_F_PULLB     0x2000u  /* blocking pread: the host reads into its host-mapped bounce,
                                     returns the range's device address in args[1], and the caller
                                     (its work-group) copies it out, then sets the slot free (B13)  */
#define GSYS_F_DEFER     0x4000u  /* non-blocking pread into device memory: the host reads into a
                                     host-mapped range and leaves a deferred-pull record; a token
                                     wait or gsys_wait's flush kernel copies it (reading B15)      */

/* Syscall numbers served (Linux x86-64). */
#define GSYS_NR_PREAD64        17
#define GSYS_NR_PWRITE64       18
#define GSYS_NR_MADVISE        28
#define GSYS_NR_SENDTO         44
#define GSYS_NR_RECVFROM       45
#define GSYS_NR_GETRUSAGE      98
#define GSYS_NR_RT_SIGQUEUEINFO 129

#define GSYS_INLINE_BYTES 256u     /* per-slot inline payload (struct rusage = 144 B)  */
#define GSYS_PREAD_CAP 0x7ffff000ull   /* Linux per-call read cap (reading A11)        */

/* ---------------------------------------------------------------- lifecycle
 * gsys_init: create the instance for the current CUDA device.
 *   slots             number of syscall-area slots; 0 = one per resident work-item of the
 *                     device ("one slot for each active GPU work-item", PAPER.md:24 P24.1),
 *                     i.e. nsmid x 2048.  Must be <= 2^24.
 *   coalesce_window_us  coalescing time window in microseconds ("a time window length within
 *                     which the CPU coalesces system calls", PAPER.md:22 P22.13); 0 = take only
 *                     requests already present.
 * Service thread count: env GSYS_THREADS (default min(16, cores-2)); coalescing max count
 * default 8 (PAPER.md:28 P28.17), see gsys_set_coalesce_max().
 * Errors: -EINVAL (slots > 2^24), -EALREADY (already initialised on this device), -ENODEV (no
 * CUDA device), -ENOMEM (pinned/device allocation failed), -ENOTSUP (stream memory operations
 * unavailable). */
int gsys_init(uint32_t slots, uint32_t coalesce_window_us);

/* Maximum number of requests one coalesced bundle may hold ("the maximum number of system call
 * invocations that can be coalesced within the time window", PAPER.md:22 P22.13).  n >= 1;
 * 1 disables coalescing.  -EINVAL for n == 0 or n > 4096, -ENODEV before gsys_init. */
int gsys_set_coalesce_max(uint32_t n);

/* Coalescing window in microseconds (same meaning as gsys_init's argument). */
int gsys_set_coalesce_window(uint32_t us);

/* Merge preads of one regular file whose ranges are adjacent or overlapping into one read of
 * the union inside a coalesced bundle (north_star extension, reading A8). on = 0/1. */
int gsys_set_merge(int on);

/* Fault injection for tests (SURVEY.md sec. 5 "failure detection"): from now on every pread whose
 * offset equals `offset` completes with -err without being executed (err 0 turns it off).  The
 * GPU caller sees the POSIX error convention of reading A4/A11.  0, -ENODEV, -EINVAL. */
int gsys_set_fault(int32_t err, int64_t offset);

/* How blocking calls on device buffers complete (env GSYS_COMPLETION=memop|host|pull at init):
 *   GSYS_COMPLETION_MEMOP -- payload by copy-engine DMA from the worker's pinned bounce,
 *       completion word in device memory written by a stream memory operation after it;
 *   GSYS_COMPLETION_HOST  -- the same DMA, then the worker waits for it and stores the host-mapped
 *       completion word;
 *   GSYS_COMPLETION_PULL (default) -- (reading B13) work-group preads that fit no pull area are read into the
 *       worker's host-mapped bounce and copied out by the work-group itself; the service makes no
 *       CUDA call while kernels wait (profiler-safe); other calls as HOST.
 * Synchronises the device first (running kernels read the setting).  0, -ENODEV, -EINVAL, -EIO. */
#define GSYS_COMPLETION_MEMOP 0u
#define GSYS_COMPLETION_HOST  1u
#define GSYS_COMPLETION_PULL  2u
int gsys_set_completion(uint32_t mode);

/* Fault injection for tests: from now on every pread whose offset equals `offset` is drained and
 * executed but its completion is never written (a lost completion); -1 turns it off.  The GPU
 * caller's watchdog (gsys_set_poll_timeout) then returns -ETIMEDOUT.  0, -ENODEV. */
int gsys_set_fault_drop(int64_t offset);

/* Watchdog (SURVEY.md sec. 5 "failure detection"; PAPER.md:30 P30.0 GPU timeouts, PAPER.md:22
 * P22.0 "raise an alarm"): every GPU-side wait on the host -- the slot claim, the completion poll,
 * a kernel-scope result, gsys_wait_token -- gives up after `ms` milliseconds (0 = never; default
 * env GSYS_POLL_TIMEOUT_MS, else 20000) and the call returns -ETIMEDOUT.  The expired wait is
 * logged on the device; the next gsys_wait() returns -ETIMEDOUT, copies the log (read it with
 * gsys_watchdog_read) and, once the service has drained, returns the affected slots to free.
 * Synchronises the device first (running kernels read the setting).  0, -ENODEV, -EIO. */
int gsys_set_poll_timeout(uint32_t ms);

/* The watchdog log as the last gsys_wait() that returned -ETIMEDOUT read it: *count expired waits
 * and up to cap records of 4 u32 {slot, seq, nr, phase (1 claim, 2 previous non-blocking request,
 * 3 completion, 4 kernel-scope result, 5 token)}.  Returns the number of records copied. */
int gsys_watchdog_read(uint32_t* count, uint32_t* recs, uint32_t cap);

/* Phase diagnostics of blocking GPU calls (enabled with env GSYS_DIAG_PHASES=1 at gsys_init):
 * out8 = {ns claiming, ns marshalling + publishing, ns waiting for completion, -, calls,
 * ns of learned pre-poll sleep, completion polls, ns copying results + releasing}, summed over
 * calls since the last reset.  0, -ENOTSUP (not enabled), -ENODEV, -EINVAL, -EIO. */
int gsys_diag_phases(uint64_t* out8, int reset);

/* Protocol tracing (debug): on = 1 records every slot transition (GPU and host side) into
 * trace buffers readable with gsys_trace_read(); capacity = max records per side. */
int gsys_set_trace(int on, uint32_t capacity);

/* Launch a kernel that may call gsys_* device functions: gsys_launch_begin(), then
 * cudaLaunchKernel(kernel, grid, block, args, smem_bytes, stream).  `kernel` is a __global__
 * function registered with libgsys's own (static) CUDA runtime -- i.e. compiled into libgsys; for a
 * kernel compiled elsewhere use gsys_launch_cu().  `args` is its argument array, `stream` a
 * cudaStream_t (NULL = the legacy default stream).  CUDA errors map to -EINVAL / -ENOMEM / -EIO. */
int gsys_launch(const void* kernel, uint32_t gx, uint32_t gy, uint32_t gz,
                uint32_t bx, uint32_t by, uint32_t bz, void** args, size_t smem_bytes,
                void* stream);

/* The same for any kernel that includes gsys_device.cuh, compiled in another module: cu_function
 * is its CUfunction (cudaGetFuncBySymbol in the caller's runtime, or cuModuleGetFunction); the
 * launch goes through the driver API (cuLaunchKernel), which every runtime shares. */
int gsys_launch_cu(void* cu_function, uint32_t gx, uint32_t gy, uint32_t gz,
                   uint32_t bx, uint32_t by, uint32_t bz, void** args, size_t smem_bytes,
                   void* stream);

/* What gsys_launch does before the launch, for callers that launch themselves (any API, CUDA
 * graphs included): reset the kernel-scope call-site records for a grid of `nblocks` blocks on
 * `stream` (they are per instance: kernel-granularity calls of launches running concurrently on
 * other streams are not supported), reset the learned completion-poll sleep, wake the service.
 * 0, -ENODEV, -EINVAL (nblocks 0 or > 2^31), -ENOMEM. */
int gsys_launch_begin(uint64_t nblocks, void* stream);

/* Drain (sec. IX "a new function call, invoked by the CPU, that ensures all GPU
 * system calls have completed before the termination of the process", P34.9).  Waits for the
 * stream (NULL = whole device), then until every request the device has published is processed
 * and its completion (DMA + state write) has landed, including the deferred pulls of non-blocking
 * device-buffer preads that no gsys_wait_token() or slot claim consumed (reading B15: one flush
 * kernel copies them all, in request order).  Returns 0, or the first -errno recorded for a
 * non-blocking call since the previous gsys_wait (reading A4), which it then clears. */
int gsys_wait(void* stream);

/* gsys_wait(NULL), stop the service threads, free everything.  Idempotent: 0 if not initialised. */
int gsys_shutdown(void);

/* Device pointer to the instance's gsys_dev_ctx (see gsys_device.cuh); NULL before init. */
const void* gsys_device_ctx(void);

/* ---------------------------------------------------------------- statistics */
typedef struct gsys_stats {
    uint64_t requests;        /* requests drained from the doorbell ring         */
    uint64_t completed;       /* requests whose completion was issued            */
    uint64_t bundles;         /* coalesced bundles handed to workers (P22.9-13)  */
    uint64_t max_bundle;      /* largest bundle seen                             */
    uint64_t host_preads;     /* pread(2) calls actually executed on the host    */
    uint64_t merged;          /* requests served by a merged union read          */
    uint64_t bytes_read;      /* bytes returned by host preads                   */
    uint64_t bytes_h2d;       /* bytes DMA'd host -> device                      */
    uint64_t errors;          /* requests that returned -errno                   */
    uint64_t per_nr[8];       /* pread, pwrite, madvise, sendto, recvfrom, getrusage, sigq, other */
    uint64_t ns_busy;         /* worker time spent processing bundles (sum over workers)   */
    uint64_t ns_syscall;      /* ... of which inside the POSIX calls themselves             */
    uint64_t ns_cuda;         /* ... of which in CUDA API calls (copies, memops, events)    */
    uint64_t ns_bounce_wait;  /* ... of which waiting for bounce-ring DMA to drain          */
    uint32_t threads;         /* service worker threads                          */
    uint32_t slots;           /* syscall-area slots                              */
    uint32_t coalesce_max;
    uint32_t coalesce_window_us;
    uint64_t split;           /* preads served in pieces by several workers (B14) */
    uint64_t deferred;        /* non-blocking preads served as deferred pulls (B15) */
    uint64_t flushed;         /* ... of which landed by gsys_wait's flush kernel   */
} gsys_stats_t;

int gsys_stats(gsys_stats_t* out);
int gsys_stats_reset(void);

/* Trace record: one slot transition ((req, slot, from, to, actor, t); the
 * validator is oracle/protocol.py check_trace).  The request is identified by (slot, seq).
 * t_ns is taken where the transition becomes visible to the other actor -- after the observation
 * it depends on (a claim after the slot was seen free, a host PROCESSING after its cmp-swap saw
 * READY) and before the store that hands the slot on (READY before the doorbell, FINISHED / FREE
 * before the completion word) -- so causal order implies timestamp order.  GPU records carry
 * %globaltimer, host records CLOCK_MONOTONIC; gsys_clock_sync() relates the two. */
typedef struct gsys_trace_rec {
    uint32_t slot;
    uint32_t seq;
    uint8_t from, to;   /* gsys_state values, `from` as observed by the actor */
    uint8_t actor;      /* 0 = GPU, 1 = host                                   */
    uint8_t blocking;   /* 1 if the request was blocking                       */
    uint32_t nr;        /* syscall number of the request                       */
    uint64_t t_ns;      /* GPU: %globaltimer; host: CLOCK_MONOTONIC            */
} gsys_trace_rec;

/* Copy up to cap records of each side into gpu_out / host_out (host memory); returns the
 * counts through n_gpu / n_host and resets the buffers. */
int gsys_trace_read(gsys_trace_rec* gpu_out, uint32_t gpu_cap, uint32_t* n_gpu,
                    gsys_trace_rec* host_out, uint32_t host_cap, uint32_t* n_host);

/* Relate the GPU's %globaltimer to the host's CLOCK_MONOTONIC: `samples` (1..4096) ping-pongs
 * between one GPU thread and the calling host thread through host-mapped words; for the sample
 * with the shortest round trip, host_time = gpu_time + *offset_ns within +- *uncertainty_ns
 * (half that round trip plus the measured %globaltimer tick).  Runs a one-thread kernel on the
 * instance's control stream.  0, -ENODEV before gsys_init, -EINVAL, -ETIMEDOUT (no answer in 1 s),
 * -EIO. */
int gsys_clock_sync(uint32_t samples, int64_t* offset_ns, uint64_t* uncertainty_ns);

/* Compile-time facts of this build, for tests: slot bytes, inline bytes, state count. */
int gsys_abi_info(uint32_t* slot_bytes, uint32_t* inline_bytes, uint32_t* nstates);

/* ---------------------------------------------------------------- host-side planning (pure)
 * The coalescer's merge planner, exported for CPU tests (no device needed).  Given n preads
 * (fd, off, len) of one bundle, computes the (fd, off) order (reading A8), groups runs on the
 * same fd whose ranges are adjacent or overlapping (off_{i+1} <= off_i + len_i) while the union
 * stays <= max_union bytes, and writes for each request its group id and its byte offset inside
 * the group's union read; group_off/group_len receive each group's union.  Returns the number
 * of groups.  order[] receives the processing order. */
int gsys_plan_merge(uint32_t n, const int32_t* fd, const int64_t* off, const uint64_t* len,
                    uint64_t max_union, uint32_t* order, uint32_t* group, uint64_t* offset_in_group,
                    int64_t* group_off, uint64_t* group_len);

/* Per-request result of a merged union read that returned r bytes (or -errno):
 * clamp(r - offset_in_group, 0, len) (reading A8); -errno propagates. */
int64_t gsys_split_result(int64_t r, uint64_t offset_in_group, uint64_t len);

/* Self-test of a worker's pinned bounce-ring allocator (host logic, no device): `iters` random
 * allocations of up to `cap` bytes with random commit points against a fake completion model;
 * checks that no allocation overlaps a region whose DMA may still be in flight.  0 or -EPROTO. */
int gsys_selftest_bounce(uint64_t seed, uint32_t iters, uint64_t cap);

/* ---------------------------------------------------------------- workloads (the hot path) */
#define GSYS_STAGE_DEVICE 0u
#define GSYS_STAGE_HOST   1u
/* Mixed: chunk k lands in a device line when (k mod 16) < n (copy-engine DMA), else in a host line
 * (SM zero-copy reads); both engines then share the host link.  n in 1..15. */
#define GSYS_STAGE_MIXED(n) (0x100u | ((n) & 15u))
/*
 * Wordcount + grep -F -l over files read with GPU-issued preads (sec. VIII-C,
 * P32.3-9 wordcount "64 strings", "work-group granularity with blocking and weak-ordering";
 * PAPER.md:30 P30.27-38 grep -F -l).
 *   fds, sizes      host arrays [nfiles]: open read-only descriptors and their sizes in bytes.
 *   chunk           bytes per work-group chunk (multiple of 16, >= 4096); each chunk [s, e) is
 *                   read with one work-group pread of [max(s-1,0), e+16) (reading A10).
 *   dict, dlen      host arrays: ndict (<= 64) words, 17-byte stride, lengths 1..16.
 *   pats, plen      host arrays: npat (<= 8) grep patterns, 17-byte stride, lengths 1..16.
 *   d_hist          DEVICE uint64[ndict]: whole-token counts are ADDED (reading A9); may be NULL when ndict == 0.
 *   d_file_hits     DEVICE uint32[nfiles] (may be NULL): set to 1 for files containing a pattern.
 *   gflags          GSYS_WG (the paper's configuration for wordcount) + GSYS_STRONG or
 *                   GSYS_RELAXED, and GSYS_BLOCKING (one pread, then the scan) or GSYS_NONBLOCKING
 *                   (each work-group prefetches its next chunk into a second line with a
 *                   non-blocking pread before scanning the current one; the slot's one-request
 *                   rule orders them, reading A15; per-chunk returns are 0 and errors surface at
 *                   gsys_wait, reading A4); another granularity is -EINVAL.
 *   staging         GSYS_STAGE_DEVICE: each work-group's pread lands in a device (HBM) line,
 *                   the host service DMAs it from its pinned bounce ring;  GSYS_STAGE_HOST: the
 *                   pread lands in a pinned host-mapped line ("syscall buffers" in system memory,
 *                   PAPER.md:24 P24.37-51) and the scan reads it over PCIe (zero-copy);
 *                   GSYS_STAGE_MIXED(n): n of every 16 chunks (by global chunk index) take the
 *                   device path, the rest the host path (each work-group owns one line of each).
 *   blocks          work-groups launched (0 = 2 per SM); threads: threads per work-group
 *                   (0 = 256; multiple of 32, <= 256).
 *   d_req_ret       DEVICE int64[total chunks] (may be NULL): per-chunk pread return value.
 *   stream          cudaStream_t to launch on.
 * Asynchronous on `stream`; call gsys_wait(stream) before reading results.  Launches share the
 * instance's workspace (chunk queue, uploads, staging lines): a call waits on the device for the
 * previous call's kernel, on whatever stream it ran, so calls on different streams serialise
 * rather than race.  Errors: -EINVAL
 * for bad sizes/flags, -ENODEV before gsys_init, CUDA errors as in gsys_launch.  Read errors
 * of individual chunks are visible in d_req_ret (negative) and skip the chunk's scan. */
int gsys_wordcount(const int32_t* fds, const uint64_t* sizes, uint32_t nfiles, uint32_t chunk,
                   const char* dict, const uint8_t* dlen, uint32_t ndict,
                   const char* pats, const uint8_t* plen, uint32_t npat,
                   uint64_t* d_hist, uint32_t* d_file_hits, int64_t* d_req_ret,
                   uint32_t gflags, uint32_t staging, uint32_t blocks, uint32_t threads, void* stream);

/* Same scan over text already resident in device memory (no syscalls): the standalone scan
 * kernel measured against the HBM roofline.  d_text: DEVICE bytes [n] (16-byte aligned); file
 * boundaries are not modelled (one file).  Adds into d_hist (NULL allowed when ndict == 0); d_hit (may be NULL) set to 1 if any
 * pattern occurs.  chunk: multiple of 16; blocks 0 = one full wave; threads 0 = 1024 (704 for
 * GSYS_SCAN_DFA_TMA), else a
 * multiple of 32 up to 1024 (768 for GSYS_SCAN_DFA_TMA); the DFA's 129-column table is used when it
 * fits beside the warps' staging, else the 77-column one.  The DFA stages each warp tile of whole
 * 64-byte rows by one swizzled tensor copy (a tensor map of d_text built per call; env
 * GSYS_SCAN_SWZ=0 at load: per-lane copies).  -EINVAL on bad
 * sizes/alignment, -ENODEV before gsys_init. */
int gsys_scan_device(const uint8_t* d_text, uint64_t n, uint32_t chunk,
                     const char* dict, const uint8_t* dlen, uint32_t ndict,
                     const char* pats, const uint8_t* plen, uint32_t npat,
                     uint64_t* d_hist, uint32_t* d_hit, uint32_t blocks, uint32_t threads,
                     void* stream);

/* Scan implementation used by gsys_wordcount and gsys_scan_device (row a8; both exact, reading
 * A9/A10): GSYS_SCAN_DFA (default) -- one transposed-DFA shared-memory lookup per byte
 * (csrc/scan_core.cuh); GSYS_SCAN_TOKEN -- SWAR word-byte masks, a per-tile list of token
 * starts, then per-token hash lookup and byte-exact verify spread over the warp
 * (csrc/tokscan.cuh; no 512-state trie limit, 0.78 of the DFA's rate on B200).  Env GSYS_SCAN=dfa|token|dfa_tma at load.  Returns the previous implementation, -EINVAL
 * for another value. */
#define GSYS_SCAN_TOKEN 0
#define GSYS_SCAN_DFA   1
#define GSYS_SCAN_DFA_TMA 2   /* gsys_scan_device: the DFA scan with bulk-copy (TMA) staging of its
                                 tiles (slower on B200; the wordcount treats it as GSYS_SCAN_DFA) */
int gsys_set_scan(int impl);

/* Diagnostics: when on, gsys_wordcount's work-groups accumulate (thread 0, %globaltimer) the
 * time spent inside their gsys_pread calls, the time spent scanning, and the chunk count;
 * gsys_read_profile copies {wait_ns, scan_ns, chunks} to host memory (optionally resetting). */
int gsys_set_profile(int on);
int gsys_read_profile(uint64_t* out3, int reset);

/* Syscall microbenchmark (sec. VII, Fig. 7/8/10): every caller of the chosen
 * granularity (work-item: every thread; work-group: every block; kernel: one per launch) issues
 * `iters` calls of
 *   kind 0 = getrusage(RUSAGE_SELF, ru) -- the blocking result lands in the slot's inline line
 *            and is copied by the caller;
 *   kind 1 = pread(fd, d_buf + caller*len, len, off), off = ((caller*iters + r) * len) mod size;
 *            after the call every thread of the calling scope reads the buffer back and the
 *            scope's byte sum is stored in d_sum[caller*iters + r] (a missing post-call barrier
 *            or an unordered DMA shows up there);
 *   kind 2 = pwrite(fd, d_buf + caller*len, len, off) after every thread of the scope wrote its
 *            share of the buffer (byte i of call idx = (idx*131 + i*7 + 13) & 0xff, written
 *            with thread-dependent delays, so a missing pre-call barrier shows up in the file).
 * d_buf: DEVICE or host-mapped, callers*len bytes (NULL allowed for kind 0).  gflags:
 * granularity + blocking + ordering.  d_ret / d_lat_ns / d_sum (each may be NULL): DEVICE
 * int64 / uint64 / uint64 [callers*iters]: return value, GPU-observed latency (ns, %globaltimer,
 * call entry -> return), and the kind-1 byte sum.  Asynchronous; returns the number of callers. */
int gsys_bench_calls(uint32_t kind, uint32_t gflags, uint32_t blocks, uint32_t threads,
                     uint32_t iters, int32_t fd, uint64_t len, uint64_t size, void* d_buf,
                     int64_t* d_ret, uint64_t* d_lat_ns, uint64_t* d_sum, void* stream);

/* ---------------------------------------------------------------- next rows
 * Config 5a -- memory management (sec. VIII-A, miniamr): one work-group per mesh
 * block, `iters` iterations.  Each iteration a work-group smooths its slice of d_field ([2][nblocks]
 * [field_words] floats, ping-pong), reads the resident set size with a GPU-issued pread of
 * statm_fd (= open("/proc/self/statm"); statm_buf: pinned host-mapped [nblocks][128] bytes) and
 * getrusage(RUSAGE_SELF), and, when d_levels[t][b] == 0 (block coarsened) and RSS >=
 * watermark_bytes, releases the host mirror [host_mesh + b*block_bytes, +block_bytes) with
 * madvise(MADV_DONTNEED) at work-group granularity with `gflags` (paper: GSYS_WG |
 * GSYS_NONBLOCKING | GSYS_RELAXED), once per block.  Outputs (DEVICE): d_released[b] = t+1 of
 * the release (0 = kept), d_rss[t] = resident bytes and d_maxrss[t] = ru_maxrss (KiB) seen by
 * work-group 0.  host_mesh must be private anonymous, page-aligned, pageable (not pinned)
 * memory.  Asynchronous; gsys_wait() surfaces madvise errors.  -EINVAL on bad arguments. */
int gsys_amr_release(uint64_t host_mesh, uint32_t nblocks, uint64_t block_bytes, const uint8_t* d_levels,
                     uint32_t iters, int32_t statm_fd, uint64_t watermark_bytes, uint64_t page_bytes,
                     float* d_field, uint32_t field_words, uint8_t* statm_buf, uint32_t* d_released,
                     int64_t* d_rss, int64_t* d_maxrss, uint32_t gflags, void* stream);

/* Config 5b -- signals (sec. VIII-B, signal-search): work-group b counts the
 * (overlapping) occurrences of key[0..keylen) (keylen 1..16) in block b of d_data ([nblocks]
 * [block_bytes], DEVICE), stores the count in counts[b] (host-mapped or device), then calls
 * rt_sigqueueinfo(tgid, sig, {si_signo = sig, si_code = SI_QUEUE, si_pid = tgid, si_uid = uid,
 * si_value.sival_int = b}) with `gflags` (paper: GSYS_WG | GSYS_NONBLOCKING).  The caller must
 * block `sig` in every thread and consume it with sigwaitinfo (libgsys's own service threads
 * block all asynchronous signals).  Asynchronous; -EINVAL on bad arguments. */
int gsys_signal_search(const uint8_t* d_data, uint32_t nblocks, uint64_t block_bytes, const uint8_t* key,
                       uint32_t keylen, int32_t tgid, int32_t sig, int32_t uid, uint32_t* counts,
                       uint32_t gflags, void* stream);

/* Config 4 -- memcached-style UDP GET server (sec. VIII-D).  gsys_mc_build lays the
 * key/value set out for the GPU: n keys (1..32 B, key_len[i] bytes at keys+key_off[i]) and values
 * (<= 4096 B at vals+val_off[i]) go to FNV-1a buckets of bucket_cap entries: d_entries (DEVICE,
 * gsys_mc_entries_bytes(nbuckets, bucket_cap) bytes), d_bucket_n (DEVICE u32[nbuckets]) and
 * d_heap (DEVICE, heap_bytes >= max(val_off+val_len)).  -E2BIG when a bucket overflows.
 * gsys_mc_serve launches nwg work-groups that loop recvfrom(fd) -> lookup -> sendto with the
 * memcached binary protocol over UDP (8-byte frame header; GET hit: status 0, 4-byte flags +
 * value; miss: status 1 + "Not found"), both calls WG-granularity: recvfrom with `gflags`
 * (blocking; paper: weak ordering), sendto with `send_gflags` (paper: blocking + weak;
 * GSYS_NONBLOCKING lets the work-group take the next request while the reply is sent).  io: pinned host-mapped [nwg][8192] request/reply buffers; stop: host-mapped
 * u32 the host sets to 1 to end the server (checked whenever recvfrom times out -- set
 * SO_RCVTIMEO on fd); d_stats (DEVICE u64[4]): served, misses, malformed, receive timeouts.
 * Keep nwg below the service thread count: each waiting recvfrom occupies a service thread. */
uint64_t gsys_mc_entries_bytes(uint32_t nbuckets, uint32_t bucket_cap);
int gsys_mc_build(const uint8_t* keys, const uint32_t* key_off, const uint8_t* key_len, const uint8_t* vals,
                  const uint64_t* val_off, const uint32_t* val_len, uint32_t n, uint32_t nbuckets,
                  uint32_t bucket_cap, void* d_entries, uint32_t* d_bucket_n, uint8_t* d_heap,
                  uint64_t heap_bytes);
int gsys_mc_serve(int32_t fd, const void* d_entries, const uint32_t* d_bucket_n, const uint8_t* d_heap,
                  uint32_t nbuckets, uint32_t bucket_cap, uint32_t nwg, uint8_t* io, const uint32_t* stop,
                  uint64_t* d_stats, uint32_t gflags, uint32_t send_gflags, void* stream);

/* Row f3 -- Fig. 8 study (sec. VII): `grid` work-groups of 1024 work-items each take
 * blocks of d_in ([nblocks][block_bytes], DEVICE, block_bytes % 16 == 0, <= 16384), apply the
 * permutation out[i] = in[d_perm[i]] `iters` times in shared memory, store the result in
 * staging[blk] (pinned host-mapped [nblocks][block_bytes]; one line per block so a non-blocking
 * write never races the next block) and pwrite it to fd at file_off + blk*block_bytes with
 * `gflags` (GSYS_WG + blocking/non-blocking + strong/relaxed).  grid 0 = one work-group per block.
 * Asynchronous; gsys_wait() drains the writes. */
int gsys_perm_pwrite(const uint8_t* d_in, const uint16_t* d_perm, uint32_t nblocks, uint32_t block_bytes,
                     uint32_t iters, uint8_t* staging, int32_t fd, uint64_t file_off, uint32_t gflags,
                     uint32_t grid, void* stream);

/* Row f4 -- Fig. 9 study (sec. VII, polling contention): nthreads GPU threads poll
 * nlines distinct 64 B lines of `lines` (pinned host-mapped or DEVICE memory, nlines*64 bytes; the
 * first u64 of each line is read) for `ns` nanoseconds with system-scope loads; d_sink (DEVICE
 * u64[2]): [0] += total polls, [1] = max(value seen) -- a host store made during the storm must be
 * observed.  Used to measure how completion polling degrades host memory throughput. */
int gsys_poll_storm(const void* lines, uint32_t nlines, uint32_t nthreads, uint64_t ns, uint64_t* d_sink,
                    void* stream);

/* Host-side consumer for GPU-issued signals: installs an async-signal-safe SA_SIGINFO handler
 * for `sig` (SIGRTMIN..SIGRTMAX) that appends si_value.sival_int to a ring of `capacity` entries
 * (any thread of the process may take the signal); gsys_sigsink_read drains up to cap values
 * (and CLOCK_MONOTONIC arrival times, t_ns may be NULL) and returns how many it copied.
 * -EINVAL for a non-real-time signal, -ENODEV before install. */
int gsys_sigsink_install(int32_t sig, uint32_t capacity);
int gsys_sigsink_read(int32_t* values, uint64_t* t_ns, uint32_t cap);

#ifdef __cplusplus
}
#endif
#endif /* GSYS_H */
