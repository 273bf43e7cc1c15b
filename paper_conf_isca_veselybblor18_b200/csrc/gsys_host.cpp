// gsys_host.cpp -- host half of libgsys: syscall area, doorbell drain, coalescing, execution.
//
// Replaces GENESYS's kernel-side processing (sec. VI "CPU-side system call
// processing", P24.16-35) with a user-space service, because the box's kernel cannot be changed
// (BASELINE.json north_star):
//   * the paper's interrupt handler ("creates a new kernel task and adds it to Linux's
//     work-queue" after "waiting for a predetermined amount of time" to coalesce, P24.17-18,
//     P24.29-30) and its OS worker thread ("atomically switches any ready system call requests to
//     the processing state" and "carries out the system call work", P24.19-21) become a pool of
//     worker threads that poll the doorbell ring the GPU writes (the s_sendmsg analogue, P24.14).
//     A free worker claims the run of ready entries at the ring head -- at most coalesce_max, and
//     it keeps extending the run for up to coalesce_window microseconds (P22.9-13) -- so bundles
//     grow by themselves when the service is the bottleneck;
//   * a bundle executes in (fd, offset) order (reading A8), preads of adjacent/overlapping ranges
//     of one regular file are merged into one read of the union (north_star extension), payloads
//     for device buffers go through a pinned bounce ring and per-bundle async copies (runs that are
//     contiguous on both sides go as one copy),
//     payloads for host-mapped buffers are read in place (P24.32-35);
//   * results go back as a completion word {seq, ret} (P24.32-34): a plain host store into pinned
//     host-mapped memory that the GPU polls (system-memory buffers, inline results and every
//     non-blocking call), or a CUDA stream memory operation ordered after the payload DMA into
//     device memory (blocking calls on device buffers);
//   * gsys_wait() is the paper's drain function (sec. IX, P34.9).
// Context fix-ups (P24.22-28) are unnecessary: the service runs inside the invoking process.

#include <cuda.h>
#include <cuda_runtime.h>
#include <errno.h>
#include <fcntl.h>
#include <immintrin.h>
#include <pthread.h>
#include <sched.h>
#include <signal.h>
#include <string.h>
#include <sys/mman.h>
#include <sys/resource.h>
#include <sys/socket.h>
#include <sys/stat.h>
#include <sys/syscall.h>
#include <time.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <deque>
#include <memory>
#include <mutex>
#include <numeric>
#include <thread>
#include <unordered_map>
#include <unordered_set>
#include <vector>

#include "gsys.h"
#include "gsys_device.cuh"
#include "gsys_internal.h"

int preload_flush_kernel();   // below, next to the flush kernel

namespace {

typedef CUresult (*PFN_batch_t)(CUstream, unsigned int, CUstreamBatchMemOpParams*, unsigned int);
typedef CUresult (*PFN_ptrattrs_t)(unsigned int, CUpointer_attribute*, void**, CUdeviceptr);
typedef CUresult (*PFN_devattr_t)(int*, CUdevice_attribute, CUdevice);
typedef CUresult (*PFN_launch_t)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                                 CUstream, void**, void**);
typedef CUresult (*PFN_funcsetattr_t)(CUfunction, CUfunction_attribute, int);

PFN_batch_t p_batch = nullptr;
PFN_ptrattrs_t p_ptrattrs = nullptr;
PFN_devattr_t p_devattr = nullptr;
PFN_launch_t p_launch = nullptr;
PFN_funcsetattr_t p_funcsetattr = nullptr;

inline uint64_t now_ns() {
    struct timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
}

int cuda_err(cudaError_t e) {
    if (e == cudaSuccess) return 0;
    if (e == cudaErrorMemoryAllocation) return -ENOMEM;
    if (e == cudaErrorInvalidValue || e == cudaErrorInvalidDeviceFunction ||
        e == cudaErrorInvalidConfiguration || e == cudaErrorInvalidResourceHandle)
        return -EINVAL;
    if (e == cudaErrorNoDevice || e == cudaErrorInvalidDevice || e == cudaErrorInsufficientDriver) return -ENODEV;
    return -EIO;
}

// ------------------------------------------------------------------ bounce ring allocator
// Ring allocator over [0, cap) of a worker's pinned bounce buffer.  Regions are handed out in
// order; a region stays "in flight" until the completion token recorded after its DMA has fired.
// alloc() waits for exactly the in-flight regions that overlap the new range: the previous lap's
// tail when it wraps, then the oldest regions of the current lap.  Ops supplies
// make_token() (flush queued copies + record an event), wait(token) and recycle(token); the
// self-test below drives it with a fake Ops.
template <class Token, class Ops>
class BounceRing {
   public:
    static constexpr size_t NONE = ~(size_t)0;
    BounceRing(size_t cap, Ops* ops) : cap_(cap), ops_(ops) {}
    size_t alloc(size_t n) {
        n = (n + 255) & ~(size_t)255;
        if (n == 0) n = 256;
        if (n > cap_) return NONE;
        if (head_ + n > cap_) {                 // wrap: retire what is left of the previous lap
            while (!q_.empty() && q_.front().lo >= head_) retire_front();
            head_ = 0;
        }
        const size_t lo = head_, hi = head_ + n;
        while (!q_.empty() && q_.front().lo < hi && lo < q_.front().hi) retire_front();
        q_.push_back(Region{lo, hi, Token{}, false, false});
        npending_++;
        head_ = hi;
        return lo;
    }
    // attach one completion token to every region allocated since the previous commit
    void commit() {
        if (!npending_) return;
        commit_with(ops_->make_token());
    }
    // ... or a given token (a pulled bounce range: released when its slot is set free)
    void commit_with(Token t) {
        if (!npending_) return;
        size_t first = q_.size() - npending_;
        for (size_t i = first; i < q_.size(); i++) {
            q_[i].tok = t;
            q_[i].committed = true;
            q_[i].last = (i + 1 == q_.size());
        }
        npending_ = 0;
    }
    // invariant for tests: no in-flight region other than the newest overlaps [lo, hi)
    bool disjoint_from_inflight(size_t lo, size_t hi) const {
        for (size_t i = 0; i + 1 < q_.size(); i++)
            if (q_[i].lo < hi && lo < q_[i].hi) return false;
        return true;
    }
    void drain() {
        while (!q_.empty()) retire_front();
    }
    size_t inflight() const { return q_.size(); }

   private:
    struct Region { size_t lo, hi; Token tok; bool committed, last; };
    void retire_front() {
        if (!q_.front().committed) commit();
        Region f = q_.front();
        // one wait per token: the regions of one commit share it (the driver call is not free)
        if (!waited_valid_ || !(waited_ == f.tok)) ops_->wait(f.tok);
        waited_ = f.tok;
        waited_valid_ = true;
        if (f.last) { ops_->recycle(f.tok); waited_valid_ = false; }
        q_.pop_front();
    }
    Token waited_{};
    bool waited_valid_ = false;
    size_t cap_, head_ = 0, npending_ = 0;
    Ops* ops_;
    std::deque<Region> q_;
};

enum PtrKind { PK_INVALID = 0, PK_DEVICE = 1, PK_HOST = 2 };

struct Instance;

// Statistics and completion counters are bumped by every worker for every request; one shared
// atomic per counter bounced its cache line between the 14 service threads.  Each thread adds to
// its own cache line (tl_shard: worker id + 1, 0 for every other thread); readers sum the shards.
// Counters are monotonic, so a sum that reaches a value means that many increments happened.
thread_local int tl_shard = 0;
struct Sharded {
    static constexpr int N = 32;
    struct alignas(64) Cell { std::atomic<uint64_t> v{0}; };
    Cell c[N];
    uint64_t fetch_add(uint64_t x, std::memory_order o = std::memory_order_seq_cst) {
        return c[tl_shard & (N - 1)].v.fetch_add(x, o);
    }
    uint64_t load(std::memory_order o = std::memory_order_seq_cst) const {
        uint64_t t = 0;
        for (const Cell& x : c) t += x.v.load(o);
        return t;
    }
    void store(uint64_t) { for (Cell& x : c) x.v.store(0); }
};

// CPUs the service threads may use: the process's allowed CPUs intersected with the GPU's
// /sys/bus/pci/devices/<bdf>/local_cpulist (its NUMA node), unless that leaves none.  Returns the
// count and fills *out (left empty when there is no locality information).
static int service_cpus(int dev, cpu_set_t* out) {
    CPU_ZERO(out);
    cpu_set_t allowed;
    CPU_ZERO(&allowed);
    if (sched_getaffinity(0, sizeof allowed, &allowed) != 0) return (int)std::thread::hardware_concurrency();
    const int nall = CPU_COUNT(&allowed);
    char bdf[32] = {0};
    if (cudaDeviceGetPCIBusId(bdf, sizeof bdf, dev) != cudaSuccess) return nall;
    for (char* c = bdf; *c; c++) *c = (char)((*c >= 'A' && *c <= 'F') ? *c - 'A' + 'a' : *c);
    char path[128];
    snprintf(path, sizeof path, "/sys/bus/pci/devices/%s/local_cpulist", bdf);
    FILE* f = fopen(path, "r");
    if (!f) return nall;
    char buf[4096];
    const size_t n = fread(buf, 1, sizeof buf - 1, f);
    fclose(f);
    buf[n] = 0;
    cpu_set_t local;
    CPU_ZERO(&local);
    for (char* p = buf; *p;) {   // "0-27,56-83"
        char* end;
        const long a = strtol(p, &end, 10);
        if (end == p) break;
        long b = a;
        p = end;
        if (*p == '-') b = strtol(p + 1, &p, 10);
        for (long c = a; c <= b && c < CPU_SETSIZE; c++) CPU_SET((int)c, &local);
        while (*p == ',' || *p == '\n' || *p == ' ') p++;
    }
    CPU_AND(out, &local, &allowed);
    const int k = CPU_COUNT(out);
    if (k == 0 || k == nall) {   // no locality information, or every allowed CPU is local anyway
        CPU_ZERO(out);
        return nall;
    }
    return k;
}

struct Req {
    uint32_t slot, seq, nr, flags;
    uint32_t pos;  // doorbell-ring position (names the deferred-pull record, B15)
    uint64_t a[6];
    int64_t ret;
    bool ok;
    bool dma;      // a host->device copy was queued for this request
    bool parked;   // blocking recvfrom on an empty socket: completed later by service_parked()
    bool faulted;  // fault injection (gsys_set_fault): completed with the injected -errno, not executed
    bool early;    // completion already issued inside the bundle (pulled bounce reads, reading B13)
    bool dropped;  // fault injection (gsys_set_fault_drop): drained, never completed
};

// A blocking recvfrom that found no datagram does not hold a service thread (reading B11): the
// request waits here and idle threads retry it (MSG_DONTWAIT) until a datagram arrives or the
// socket's SO_RCVTIMEO expires, so the GPU caller still sees one blocking POSIX call.
struct Parked {
    Req r;
    uint64_t deadline_ns;   // UINT64_MAX: no receive timeout
};

// A large pread served by several workers at once (reading B14): when other workers are idle, the
// worker that drained the request cuts its byte range into pieces that idle workers read in
// parallel; whoever finishes the last piece assembles the single-call POSIX result (the bytes up to
// the first short piece, or the first piece's error) and issues the completion with a host store.
// Still one request and one completion: the GPU caller sees one blocking pread.
struct Split {
    Req r;
    int fd = -1;
    uint8_t* dst = nullptr;
    int64_t off = 0;
    uint64_t n = 0, piece = 0;
    uint32_t np = 0;
    std::atomic<uint32_t> next{0};   // next piece to claim
    std::atomic<uint32_t> done{0};   // pieces finished
    std::vector<int64_t> ret;
};

// Host-mapped ranges holding deferred pulls (reading B15), handed out in ring order and recycled in
// order once their record says consumed.  alloc() never waits: when the oldest range is still
// unconsumed the caller falls back to the copy-engine path.
struct DeferRing {
    uint8_t* h = nullptr;      // pinned, mapped
    uint8_t* d = nullptr;      // its device address
    size_t cap = 0, head = 0;
    struct Region { size_t lo, hi; uint32_t pos; };
    std::deque<Region> q;
    std::mutex mu;             // q is also read by gsys_wait's flush
    gsys_nbrec* recs = nullptr;
    uint32_t mask = 0;
    bool consumed(const Region& g) const {
        const gsys_nbrec& r = recs[g.pos & mask];
        return __atomic_load_n(&r.consumed, __ATOMIC_ACQUIRE) != 0u || __atomic_load_n(&r.tag, __ATOMIC_ACQUIRE) != g.pos + 1u;
    }
    // offset of n free bytes, or ~0 (ring order: the free space runs from the newest region's end
    // to the oldest outstanding region's start)
    // Consumed regions are retired lazily -- only when the free space cannot take n bytes -- so
    // a request reads no GPU-written record line unless the ring has to make room.
    size_t alloc(size_t n, uint32_t pos) {
        n = (n + 255) & ~(size_t)255;
        if (n > cap) return ~(size_t)0;
        std::lock_guard<std::mutex> g(mu);
        size_t lo = fit(n);
        while (lo == ~(size_t)0 && !q.empty() && consumed(q.front())) {
            q.pop_front();
            lo = fit(n);
        }
        if (lo == ~(size_t)0) return lo;
        q.push_back(Region{lo, lo + n, pos});
        head = lo + n;
        return lo;
    }
    size_t fit(size_t n) const {
        if (q.empty()) return 0;
        const size_t tail = q.front().lo;
        if (head > tail) {               // not wrapped: [head, cap) then [0, tail)
            if (head + n <= cap) return head;
            if (n <= tail) return 0;
            return ~(size_t)0;
        }
        return head + n <= tail ? head : ~(size_t)0;   // wrapped: [head, tail)
    }
};

// ------------------------------------------------------------------ worker
struct Worker {
    Instance* inst = nullptr;
    int id = 0;
    std::thread th;
    cudaStream_t stream = nullptr;
    uint8_t* bounce = nullptr;       // pinned
    size_t bcap = 0;
    // BounceRing ops: a token is either a CUDA event recorded after the queued copies were issued,
    // or (pulled bounce reads, reading B13) the (slot, seq) whose work-group copies the range out
    // and then sets the slot free
    struct Tok {
        cudaEvent_t ev = nullptr;
        uint32_t slot = 0, seq = 0;
        bool operator==(const Tok& o) const { return ev == o.ev && slot == o.slot && seq == o.seq; }
    };
    struct RingOps {
        Worker* w;
        Tok make_token() {
            w->flush_copies();
            Timer t(w->t_cuda);
            Tok k;
            k.ev = w->get_event();
            cudaEventRecord(k.ev, w->stream);
            return k;
        }
        void wait(const Tok& k) {
            Timer t(w->t_wait);
            if (k.ev) { cudaEventSynchronize(k.ev); return; }
            w->wait_slot_free(k.slot, k.seq);
        }
        void recycle(const Tok& k) { if (k.ev) w->evpool.push_back(k.ev); }
    };
    RingOps ring_ops{this};
    uint64_t t_sys = 0, t_cuda = 0, t_wait = 0;   // per-bundle timers (ns)
    struct Timer {
        uint64_t& acc; uint64_t t0;
        explicit Timer(uint64_t& a) : acc(a), t0(now_ns()) {}
        ~Timer() { acc += now_ns() - t0; }
    };
    BounceRing<Tok, RingOps>* ring = nullptr;
    uint8_t* bounce_d = nullptr;     // device address of the (host-mapped) bounce
    DeferRing defer;                 // deferred pulls of non-blocking preads (B15)
    DeferRing defer2;                // overflow store, allocated the first time `defer` is full
    bool defer2_failed = false;      // its allocation failed: overflow takes the copy engine
    // destination -> ring position of the newest deferred pull this worker served into it
    // (overflow ordering).  Written by this worker only, so its lines stay in this core's cache;
    // the rare overflow reader takes every worker's lock and the newest pending entry
    std::mutex dmu;
    std::unordered_map<uint64_t, uint32_t> dmap;
    bool try_defer(Req& r, int fd, uint64_t n, int64_t off, int64_t* ret);
    void wait_slot_free(uint32_t slot, uint32_t seq);
    void complete_early(Req& r);
    bool try_split(Req& r, int fd, uint8_t* dst, uint64_t n, int64_t off);
    std::vector<cudaEvent_t> evpool;
    // copies queued per bundle; flush_copies() issues them (contiguous runs joined)
    std::vector<void*> cp_dst, cp_src;
    std::vector<size_t> cp_len;
    std::vector<Req> reqs;
    std::vector<CUstreamBatchMemOpParams> ops;
    struct Cache { uintptr_t lo, hi; PtrKind kind; intptr_t host_delta; uint64_t gen; };
    std::vector<Cache> cache;
    // merge scratch
    std::vector<int32_t> mfd; std::vector<int64_t> moff; std::vector<uint64_t> mlen;
    std::vector<uint32_t> morder, mgroup; std::vector<uint64_t> mgoff_in; std::vector<int64_t> mg_off;
    std::vector<uint64_t> mg_len; std::vector<uint32_t> midx;
    std::vector<uint8_t> done_;                        // per-bundle scratch, reused
    std::vector<std::vector<uint32_t>> members_;

    cudaEvent_t get_event() {
        if (!evpool.empty()) { cudaEvent_t e = evpool.back(); evpool.pop_back(); return e; }
        cudaEvent_t e;
        cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
        return e;
    }
    // n bytes of pinned bounce; waits for in-flight DMA still reading the range
    uint8_t* alloc(size_t n) {
        size_t o = ring->alloc(n);
        return o == ring->NONE ? nullptr : bounce + o;
    }
    void commit() { ring->commit(); }
    void flush_copies();
    PtrKind resolve(uintptr_t p, size_t n, uint8_t** host);
    void run();
    void process(uint64_t h0, uint32_t n);
    int64_t do_pread(Req& r);
    int64_t do_pwrite(Req& r);
    int64_t do_getrusage(Req& r);
    int64_t do_generic(Req& r);
    int64_t do_recvfrom(Req& r, bool may_park);
    void service_parked();
    int read_small(uintptr_t p, void* out, size_t n);
    int write_small(uintptr_t p, const void* in, size_t n);
    // queue a host->device copy; issued with the bundle's other copies by flush_copies()
    bool dma_flag = false;
    void h2d(void* dst, const void* src, size_t n) {
        dma_flag = true;
        cp_dst.push_back(dst);
        cp_src.push_back(const_cast<void*>(src));
        cp_len.push_back(n);
    }
};

// ------------------------------------------------------------------ instance
struct Instance {
    int dev = -1;
    cpu_set_t cpus;                 // service-thread CPUs (this GPU's NUMA-local ones), empty = any
    uint32_t nslots = 0;
    gsys_slot* area_h = nullptr;        // pinned, mapped
    gsys_slot* area_d = nullptr;
    uint8_t* inline_h = nullptr;
    uint8_t* pull_h = nullptr;          // pinned, mapped: [(nslots/32) * pull_bytes] (reading B12)
    uint8_t* pull_d = nullptr;
    uint32_t pull_bytes = 0;
    // host address of slot s's pull area for an n-byte pread (the device's pull_src rule), or null
    uint8_t* pull_area(uint32_t s, uint64_t n) const {
        if (n == 0) return nullptr;
        if (n <= GSYS_INLINE_BYTES) return inline_h + (size_t)s * GSYS_INLINE_BYTES;
        if ((s & 31u) == 0u && n <= pull_bytes && pull_h) return pull_h + (size_t)(s >> 5) * pull_bytes;
        return nullptr;
    }
    uint8_t* inline_d = nullptr;
    uint64_t* ring_h = nullptr;
    uint64_t* ring_d = nullptr;
    uint32_t ring_cap = 0;
    uint32_t* claim_d = nullptr;
    uint32_t* seqs_d = nullptr;
    unsigned long long* mirror_d = nullptr;
    uint64_t* hdone_h = nullptr;        // pinned, mapped: host-store completion words
    uint64_t* hdone_d = nullptr;
    uint32_t* tail_d = nullptr;
    uint32_t* lat_hint_d = nullptr;
    uint32_t* nbpend_d = nullptr;
    uint32_t* nbpos_d = nullptr;
    uint32_t* nbclaim_d = nullptr;
    gsys_kround* krounds_d = nullptr;
    uint32_t* kblock_d = nullptr;
    uint32_t kblock_cap = 0;
    std::vector<void*> graveyard;       // superseded device buffers (freed at shutdown)
    gsys_trace_rec* gtrace_d = nullptr;
    uint32_t* gtrace_n_d = nullptr;
    uint32_t trace_cap = 0;
    gsys_dev_ctx ctx_h{};
    gsys_dev_ctx* ctx_d = nullptr;
    cudaStream_t ctl = nullptr;
    bool mem64 = true;
    bool memop_completion = false;      // see gsys_dev_ctx::memop_completion
    unsigned long long* diag_d = nullptr;   // GSYS_DIAG_PHASES accumulators (device)

    // service
    std::vector<Worker*> workers;
    std::atomic<bool> stop{false};
    alignas(64) std::atomic<uint64_t> head{0};   // doorbell entries claimed by workers
    Sharded completed;                     // requests whose completion was issued
    std::atomic<int> first_err{0};
    std::atomic<uint32_t> coalesce_max{8};
    std::atomic<uint32_t> window_us{0};
    std::atomic<int> merge{1};
    std::atomic<int> fault_err{0};          // gsys_set_fault: preads at fault_off fail with -fault_err
    std::atomic<int64_t> fault_off{-1};
    std::atomic<int64_t> drop_off{-1};      // gsys_set_fault_drop: that pread's completion is never written
    // split preads (reading B14): queue of ranges with pieces left, shared by all workers
    std::mutex split_mu;
    std::deque<std::shared_ptr<Split>> splits;
    std::atomic<int> nsplits{0};
    uint64_t split_min = 128u << 10;      // env GSYS_SPLIT_KB (0 = never split)
    size_t defer_grow = 64u << 20;        // per-worker overflow store for deferred pulls, allocated
                                          // on first overflow (env GSYS_DEFER_GROW_MB, 0 = none)
    Sharded st_split;                      // preads served in pieces
    Sharded st_deferred;                   // non-blocking preads served as deferred pulls (B15)
    Sharded st_flushed;                    // ... of which copied by gsys_wait's flush
    gsys_nbrec* nbrec_h = nullptr;         // pinned, mapped [ring_cap]: deferred-pull records
    gsys_nbrec* nbrec_d = nullptr;
    // land the deferred pulls nobody has consumed yet, in request order: every one (upto_all) or
    // those at or before ring position `upto`; by one flush kernel per pass (no kernel may be
    // running: gsys_wait) or by copy-engine copies (from a service thread: an application kernel
    // may fill the GPU and wait on this service, so no SM work can be relied on)
    int flush_deferred(cudaStream_t st, bool upto_all, uint32_t upto, bool use_kernel, uint64_t only_dst = 0);
    std::mutex flush_mu;
    void* flush_buf = nullptr;             // pinned, mapped: the flush kernel's record list
    size_t flush_cap = 0;
    std::vector<void*> flush_old;
    bool run_piece(Split& sp, uint32_t i);
    bool help_split();
    gsys_wd_log* wd_d = nullptr;           // device watchdog log (gsys_device.cuh)
    std::mutex wd_mu;
    gsys_wd_log wd_last{};                 // the log as the last gsys_wait that saw expiries read it
    Sharded st_faults;
    std::atomic<uint64_t> gen{1};          // pointer-cache generation
    std::atomic<uint64_t> kick{0};
    std::atomic<int> idle_workers{0};      // workers that found the ring empty and claimed nothing since
    bool share_bursts = true;              // split a burst among idle workers (env GSYS_SHARE_BURSTS=0: off)
    bool big_alone = true;                 // preads > 64 KiB into host memory are claimed alone (env GSYS_BIG_ALONE=0: off)
    std::mutex sleep_mu;
    std::condition_variable sleep_cv;
    std::atomic<int> sleepers{0};
    std::mutex park_mu;
    std::vector<Parked> parked;
    std::atomic<uint32_t> nparked{0};
    // host-store completion (args[0], state, completion word) of a request finished outside process()
    void complete_host(const Req& r);
    uint32_t nthreads = 0;

    // stats
    Sharded st_ns_busy, st_ns_syscall, st_ns_cuda, st_ns_wait;
    Sharded st_bundles, st_host_preads, st_merged, st_bytes_read, st_bytes_h2d, st_errors;
    std::atomic<uint64_t> st_max_bundle{0};
    Sharded st_nr[8];

    // host trace
    std::atomic<int> tracing{0};
    std::mutex trace_mu;
    std::vector<gsys_trace_rec> htrace;

    Instance() {}

    // stamped after the observation the edge depends on and before the store that hands the slot
    // back (gsys.h gsys_trace_rec)
    void host_trace(uint32_t s, uint32_t seq, uint8_t from, uint8_t to, bool blocking, uint32_t nr) {
        if (!tracing.load(std::memory_order_relaxed)) return;
        std::lock_guard<std::mutex> g(trace_mu);
        if (htrace.size() < trace_cap) {
            gsys_trace_rec r;
            r.slot = s; r.seq = seq; r.from = from; r.to = to; r.actor = 1; r.blocking = blocking ? 1 : 0;
            r.nr = nr; r.t_ns = now_ns();
            htrace.push_back(r);
        }
    }
    bool ready(uint64_t pos) const {
        uint64_t v = __atomic_load_n(&ring_h[pos & (ring_cap - 1)], __ATOMIC_ACQUIRE);
        return (uint32_t)(v >> 32) == (uint32_t)(pos + 1);
    }
};

Instance* g_inst[64] = {nullptr};
std::mutex g_mu;

Instance* current() {
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess || d < 0 || d >= 64) return nullptr;
    return g_inst[d];
}

inline int nr_index(uint32_t nr) {
    switch (nr) {
        case GSYS_NR_PREAD64: return 0;
        case GSYS_NR_PWRITE64: return 1;
        case GSYS_NR_MADVISE: return 2;
        case GSYS_NR_SENDTO: return 3;
        case GSYS_NR_RECVFROM: return 4;
        case GSYS_NR_GETRUSAGE: return 5;
        case GSYS_NR_RT_SIGQUEUEINFO: return 6;
        default: return 7;
    }
}

// ------------------------------------------------------------------ worker (interrupt handler + OS worker)
void Worker::run() {
    // service threads take no asynchronous signals: a GPU-issued rt_sigqueueinfo to this process
    // must reach the application's sigwaitinfo consumer, never a worker
    sigset_t ss;
    sigfillset(&ss);
    sigdelset(&ss, SIGSEGV);
    sigdelset(&ss, SIGBUS);
    sigdelset(&ss, SIGFPE);
    sigdelset(&ss, SIGILL);
    sigdelset(&ss, SIGABRT);
    pthread_sigmask(SIG_BLOCK, &ss, nullptr);
    if (CPU_COUNT(&inst->cpus) > 0) sched_setaffinity(0, sizeof inst->cpus, &inst->cpus);   // NUMA-local
    tl_shard = id + 1;
    cudaSetDevice(inst->dev);
    Instance* I = inst;
    uint64_t idle_since = now_ns();
    uint64_t last_kick = I->kick.load();
    bool idle = false;   // counted in I->idle_workers
    while (!I->stop.load(std::memory_order_relaxed)) {
        uint64_t h = I->head.load(std::memory_order_acquire);
        if (!I->ready(h)) {
            if (!idle) { idle = true; I->idle_workers.fetch_add(1, std::memory_order_relaxed); }
            if (I->nsplits.load(std::memory_order_relaxed) && I->help_split()) {   // pieces of a split pread
                idle_since = now_ns();
                continue;
            }
            if (I->nparked.load(std::memory_order_relaxed)) {   // parked recvfroms keep us awake
                service_parked();
                idle_since = now_ns();
                _mm_pause();
                continue;
            }
            uint64_t k = I->kick.load(std::memory_order_relaxed);
            if (k != last_kick) { last_kick = k; idle_since = now_ns(); }
            if (now_ns() - idle_since > 2000000ull) {
                std::unique_lock<std::mutex> lk(I->sleep_mu);
                I->sleepers.fetch_add(1);
                I->sleep_cv.wait_for(lk, std::chrono::microseconds(50));
                I->sleepers.fetch_sub(1);
            } else {
                _mm_pause();
            }
            continue;
        }
        // claim the run of ready entries at the head (a coalesced bundle, P22.9-13)
        const uint32_t cmax = I->coalesce_max.load(std::memory_order_relaxed);
        const uint64_t win = (uint64_t)I->window_us.load(std::memory_order_relaxed) * 1000ull;
        uint32_t n = 1;
        while (n < cmax && I->ready(h + n)) n++;
        if (!win && n > 1 && I->big_alone) {
            // a large pread into host memory is never merged (reading A8: it would add a memcpy), so
            // riding in a bundle (served serially, P22.12) only holds up the requests behind it:
            // take it alone and leave its neighbours to other workers
            const gsys_slot* sl = I->area_h + (uint32_t)__atomic_load_n(&I->ring_h[h & (I->ring_cap - 1)], __ATOMIC_ACQUIRE);
            if (__atomic_load_n(&sl->nr, __ATOMIC_RELAXED) == GSYS_NR_PREAD64 &&
                (__atomic_load_n(&sl->flags, __ATOMIC_RELAXED) & GSYS_HOSTBUF) &&
                __atomic_load_n(&sl->args[2], __ATOMIC_RELAXED) > (64u << 10))
                n = 1;
        }
        if (!win && n > 1 && I->share_bursts) {
            // a bundle is served serially (P22.12): with other workers idle, share a burst among
            // them instead of serialising it here (64 simultaneous 256 KiB preads: 8 bundles of 8
            // on 8 workers would leave 6 idle); under load nobody is idle and bundles stay <= max
            const uint32_t avail = (uint32_t)I->idle_workers.load(std::memory_order_relaxed) + (idle ? 0u : 1u);
            const uint32_t share = (n + (avail ? avail : 1u) - 1u) / (avail ? avail : 1u);
            if (share < n) n = share;
        }
        if (!I->head.compare_exchange_strong(h, h + n, std::memory_order_acq_rel)) continue;
        if (idle) { idle = false; I->idle_workers.fetch_sub(1, std::memory_order_relaxed); }
        // coalescing window: keep extending the run for up to window microseconds (reading A19)
        if (win && n < cmax) {
            const uint64_t t0 = now_ns();
            while (n < cmax && now_ns() - t0 < win) {
                uint64_t e = h + n;
                if (!I->ready(e)) { _mm_pause(); continue; }
                if (!I->head.compare_exchange_strong(e, e + 1, std::memory_order_acq_rel)) break;
                n++;
            }
        }
        I->st_bundles.fetch_add(1, std::memory_order_relaxed);
        uint64_t mb = I->st_max_bundle.load(std::memory_order_relaxed);
        while (n > mb && !I->st_max_bundle.compare_exchange_weak(mb, n)) {}
        process(h, n);
        if (I->nparked.load(std::memory_order_relaxed)) service_parked();
        idle_since = now_ns();
    }
}

void Worker::flush_copies() {
    size_t n = cp_dst.size();
    if (!n) return;
    Timer tm(t_cuda);
    // one cudaMemcpyAsync per run of copies that are contiguous in both source and destination
    // (a merged union read split into neighbouring work-group lines is one such run); the batched
    // copy entry points are not used (they raised GPU faults on this pool's driver)
    size_t i = 0;
    while (i < n) {
        uint8_t* d = (uint8_t*)cp_dst[i];
        const uint8_t* sp = (const uint8_t*)cp_src[i];
        size_t len = cp_len[i];
        size_t j = i + 1;
        while (j < n && (uint8_t*)cp_dst[j] == d + len && (const uint8_t*)cp_src[j] == sp + len) len += cp_len[j++];
        cudaMemcpyAsync(d, sp, len, cudaMemcpyHostToDevice, stream);
        i = j;
    }
    cp_dst.clear();
    cp_src.clear();
    cp_len.clear();
}

// Pinned host ranges allocated by the library itself (e.g. the wordcount's zero-copy staging):
// recognised without a driver call, so the service never touches the CUDA API while serving
// system-memory buffers (which also keeps it out of a profiler's serialisation lock).
struct HostRange { std::atomic<uintptr_t> lo{0}, hi{0}; };
HostRange g_host_ranges[32];
std::atomic<int> g_nhost_ranges{0};

PtrKind Worker::resolve(uintptr_t p, size_t n, uint8_t** host) {
    const int nr = g_nhost_ranges.load(std::memory_order_acquire);
    for (int i = 0; i < nr; i++) {
        const uintptr_t lo = g_host_ranges[i].lo.load(std::memory_order_relaxed);
        const uintptr_t hi = g_host_ranges[i].hi.load(std::memory_order_relaxed);
        if (p >= lo && p + n <= hi) {
            if (host) *host = (uint8_t*)p;
            return PK_HOST;
        }
    }
    uint64_t g = inst->gen.load(std::memory_order_relaxed);
    for (auto& c : cache) {
        if (c.gen == g && p >= c.lo && p + n <= c.hi) {
            if (host) *host = (uint8_t*)(p + c.host_delta);
            return c.kind;
        }
    }
    if (p == 0) return PK_INVALID;
    CUpointer_attribute attrs[4] = {CU_POINTER_ATTRIBUTE_MEMORY_TYPE, CU_POINTER_ATTRIBUTE_RANGE_START_ADDR,
                                    CU_POINTER_ATTRIBUTE_RANGE_SIZE, CU_POINTER_ATTRIBUTE_HOST_POINTER};
    unsigned int mtype = 0;
    CUdeviceptr start = 0;
    size_t size = 0;
    void* hp = nullptr;
    void* data[4] = {&mtype, &start, &size, &hp};
    if (p_ptrattrs(4, attrs, data, (CUdeviceptr)p) != CUDA_SUCCESS) return PK_INVALID;
    PtrKind k = PK_INVALID;
    intptr_t delta = 0;
    if (mtype == CU_MEMORYTYPE_DEVICE) {
        k = PK_DEVICE;
    } else if (mtype == CU_MEMORYTYPE_HOST || mtype == CU_MEMORYTYPE_UNIFIED) {
        k = PK_HOST;
        if (hp) delta = (intptr_t)hp - (intptr_t)p;
    }
    if (k == PK_INVALID) return k;
    if (size == 0) { start = (CUdeviceptr)p; size = n; }
    if (cache.size() >= 32) cache.erase(cache.begin());
    cache.push_back(Cache{(uintptr_t)start, (uintptr_t)start + size, k, delta, g});
    if (p + n > (uintptr_t)start + size) return PK_INVALID;
    if (host) *host = (uint8_t*)(p + delta);
    return k;
}

int Worker::read_small(uintptr_t p, void* out, size_t n) {
    uint8_t* hp = nullptr;
    PtrKind k = resolve(p, n, &hp);
    if (k == PK_HOST) { memcpy(out, hp, n); return 0; }
    if (k == PK_DEVICE) {
        if (cudaMemcpyAsync(out, (void*)p, n, cudaMemcpyDeviceToHost, stream) != cudaSuccess) return -EFAULT;
        cudaStreamSynchronize(stream);
        return 0;
    }
    return -EFAULT;
}

int Worker::write_small(uintptr_t p, const void* in, size_t n) {
    uint8_t* hp = nullptr;
    PtrKind k = resolve(p, n, &hp);
    if (k == PK_HOST) { memcpy(hp, in, n); return 0; }
    if (k == PK_DEVICE) {
        uint8_t* b = alloc(n);
        if (!b) return -ENOMEM;
        memcpy(b, in, n);
        h2d((void*)p, b, n);
        return 0;
    }
    return -EFAULT;
}

// A pulled bounce range is free again once its work-group set the slot free (or the slot already
// carries a newer request).  Bounded by the watchdog timeout: a work-group that died without
// consuming its range must not wedge the worker forever.
void Worker::wait_slot_free(uint32_t slot, uint32_t seq) {
    const gsys_slot* sl = inst->area_h + slot;
    const uint64_t t0 = now_ns();
    const uint64_t lim = inst->ctx_h.poll_timeout_ns ? 2 * inst->ctx_h.poll_timeout_ns : 0;
    for (;;) {
        if (__atomic_load_n(&sl->state, __ATOMIC_ACQUIRE) == GSYS_FREE) return;
        if (__atomic_load_n(&sl->seq, __ATOMIC_ACQUIRE) != seq) return;
        if (lim && now_ns() - t0 > lim) {
            inst->st_errors.fetch_add(1, std::memory_order_relaxed);
            return;
        }
        _mm_pause();
    }
}

// Completion of one request inside its bundle (reading B13): result, state, completion word now,
// so its work-group can start copying while the rest of the bundle is served.
void Worker::complete_early(Req& r) {
    r.early = true;
    if (r.dropped) { inst->completed.fetch_add(1, std::memory_order_release); return; }
    inst->complete_host(r);
}

// Split a large pread among idle workers (reading B14).  Returns true when the request was handed
// to the split machinery: its completion is then issued by the worker that finishes the last piece.
bool Worker::try_split(Req& r, int fd, uint8_t* dst, uint64_t n, int64_t off) {
    Instance* I = inst;
    if (!I->split_min || n < I->split_min || r.dropped || r.faulted || !r.ok) return false;
    const int idle = I->idle_workers.load(std::memory_order_relaxed);
    if (idle < 1) return false;
    uint32_t np = (uint32_t)std::min<uint64_t>(std::min<uint64_t>((uint64_t)idle + 1, n / (32u << 10)), 16);
    if (np < 2) return false;
    auto sp = std::make_shared<Split>();
    sp->r = r;
    sp->fd = fd;
    sp->dst = dst;
    sp->off = off;
    sp->n = n;
    sp->piece = ((n + np - 1) / np + 4095) & ~(uint64_t)4095;
    sp->np = (uint32_t)((n + sp->piece - 1) / sp->piece);
    sp->ret.assign(sp->np, 0);
    r.early = true;   // completed by the last piece's worker
    {
        std::lock_guard<std::mutex> g(I->split_mu);
        I->splits.push_back(sp);
        I->nsplits.fetch_add(1, std::memory_order_release);
    }
    { Timer tm(t_sys); while (I->run_piece(*sp, sp->next.fetch_add(1, std::memory_order_acq_rel))) {} }
    return true;
}

// Non-blocking pread into device memory (reading B15): read into a host-mapped range and record
// {src, dst, ret} at the request's ring position before the completion is published; the bytes
// reach dst when a token wait or gsys_wait's flush copies them.  false: not deferred (host
// destination, or no free range), serve it the usual way.
bool Worker::try_defer(Req& r, int fd, uint64_t n, int64_t off, int64_t* ret) {
    if (!defer.h) return false;
    uintptr_t dst = (uintptr_t)r.a[1];
    uint8_t* hp = nullptr;
    if (resolve(dst, n, &hp) != PK_DEVICE) return false;
    uint64_t want = std::min<uint64_t>(std::min<uint64_t>(n, GSYS_PREAD_CAP), defer.cap);
    DeferRing* st = &defer;
    size_t o = defer.alloc(want, r.pos);
    if (o == ~(size_t)0 && inst->defer_grow) {
        // the store is full of pulls nobody has consumed yet (many callers, e.g. work-item
        // granularity): a second, larger store takes the overflow -- allocated once, on demand,
        // so callers that never fill the first keep its smaller, cache-friendlier footprint
        if (!defer2.h && !defer2_failed) {
            Timer tm(t_cuda);
            uint8_t* hp = nullptr;
            uint8_t* dp = nullptr;
            if (cudaHostAlloc((void**)&hp, inst->defer_grow, cudaHostAllocMapped | cudaHostAllocPortable) ==
                    cudaSuccess &&
                cudaHostGetDevicePointer((void**)&dp, hp, 0) == cudaSuccess) {
                std::lock_guard<std::mutex> g(defer2.mu);   // gsys_wait's flush reads the store under it
                defer2.recs = defer.recs;
                defer2.mask = defer.mask;
                defer2.cap = inst->defer_grow;
                defer2.d = dp;
                defer2.h = hp;
            } else {
                cudaGetLastError();
                if (hp) cudaFreeHost(hp);
                defer2_failed = true;
            }
        }
        if (defer2.h) {
            want = std::min<uint64_t>(std::min<uint64_t>(n, GSYS_PREAD_CAP), defer2.cap);
            o = defer2.alloc(want, r.pos);
            st = &defer2;
        }
    }
    if (o == ~(size_t)0) {
        // the range store is full of pulls nobody has consumed yet: this request takes the
        // copy-engine path -- after any pending pull into the same buffer has landed (by copy
        // engine, in request order), so the older read cannot overwrite this one
        uint32_t last = 0;
        bool pending = false;
        for (Worker* w : inst->workers) {
            std::lock_guard<std::mutex> g(w->dmu);
            auto it = w->dmap.find((uint64_t)dst);
            if (it == w->dmap.end()) continue;
            const gsys_nbrec& pr = inst->nbrec_h[it->second & (inst->ring_cap - 1)];
            const bool p = __atomic_load_n(&pr.tag, __ATOMIC_ACQUIRE) == it->second + 1u &&
                           !__atomic_load_n(&pr.consumed, __ATOMIC_ACQUIRE);
            if (!p) { w->dmap.erase(it); continue; }
            if (!pending || (int32_t)(it->second - last) > 0) last = it->second;
            pending = true;
        }
        if (pending) {
            Timer tm(t_cuda);
            inst->flush_deferred(stream, false, last, false, (uint64_t)dst);
        }
        return false;
    }
    ssize_t z;
    { Timer tm(t_sys); z = pread(fd, st->h + o, want, off); }
    inst->st_host_preads.fetch_add(1, std::memory_order_relaxed);
    *ret = z < 0 ? -(int64_t)errno : (int64_t)z;
    if (z > 0) inst->st_bytes_read.fetch_add((uint64_t)z, std::memory_order_relaxed);
    gsys_nbrec& rec = inst->nbrec_h[r.pos & (inst->ring_cap - 1)];
    // the record slot of this ring position still holds a pull nobody consumed (ring_cap requests
    // ago): land it (and everything older) before its record is reused
    if (__atomic_load_n(&rec.tag, __ATOMIC_ACQUIRE) == r.pos + 1u - inst->ring_cap &&
        !__atomic_load_n(&rec.consumed, __ATOMIC_ACQUIRE) && rec.src && rec.ret > 0) {
        Timer tm(t_cuda);
        inst->flush_deferred(stream, false, r.pos - inst->ring_cap, false);
    }
    __atomic_store_n(&rec.src, z > 0 ? (uint64_t)(uintptr_t)(st->d + o) : 0ull, __ATOMIC_RELAXED);
    __atomic_store_n(&rec.dst, (uint64_t)dst, __ATOMIC_RELAXED);
    __atomic_store_n(&rec.ret, (long long)*ret, __ATOMIC_RELAXED);
    __atomic_store_n(&rec.consumed, z > 0 ? 0u : 1u, __ATOMIC_RELAXED);   // nothing to copy: free at once
    __atomic_store_n(&rec.tag, r.pos + 1u, __ATOMIC_RELEASE);   // published with the completion word after it
    inst->st_deferred.fetch_add(1, std::memory_order_relaxed);
    if (z > 0) {
        std::lock_guard<std::mutex> g(dmu);
        dmap[(uint64_t)dst] = r.pos;
    }
    return true;
}

// pread(fd, buf, n, off): host-mapped buf -> read in place; device buf -> read into the pinned
// bounce and DMA.  A request larger than the bounce is served piecewise with the POSIX result of
// one call (stop at a short piece, cap at GSYS_PREAD_CAP, reading A11).
int64_t Worker::do_pread(Req& r) {
    int fd = (int)r.a[0];
    uintptr_t buf = (uintptr_t)r.a[1];
    uint64_t n = r.a[2];
    int64_t off = (int64_t)r.a[3];
    if (n == 0) {
        ssize_t z = pread(fd, nullptr, 0, off);
        return z < 0 ? -(int64_t)errno : 0;
    }
    uint8_t* hp = nullptr;
    PtrKind k;
    if (r.flags & GSYS_F_PULLB) {
        // reading B13: read into this worker's host-mapped bounce, hand the range's device address
        // back in args[1] and complete at once; the work-group copies the bytes to its buffer and
        // sets the slot free, which releases the range (no CUDA call on this path)
        const uint64_t want = std::min<uint64_t>(std::min<uint64_t>(n, GSYS_PREAD_CAP), bcap / 2);
        commit();   // earlier regions of this bundle keep their own tokens
        uint8_t* b = alloc(want);
        if (!b) return -ENOMEM;
        Worker::Tok t;
        t.slot = r.slot;
        t.seq = r.seq;
        ring->commit_with(t);
        __atomic_store_n(&inst->area_h[r.slot].args[1], (uint64_t)(uintptr_t)(bounce_d + (b - bounce)), __ATOMIC_RELAXED);
        if (try_split(r, fd, b, want, off)) return 0;
        ssize_t z;
        { Timer tm(t_sys); z = pread(fd, b, want, off); }
        inst->st_host_preads.fetch_add(1, std::memory_order_relaxed);
        r.ret = z < 0 ? -(int64_t)errno : (int64_t)z;
        if (z > 0) inst->st_bytes_read.fetch_add((uint64_t)z, std::memory_order_relaxed);
        complete_early(r);
        return r.ret;
    }
    if ((r.flags & GSYS_F_DEFER) && !r.dropped) {
        int64_t dret = 0;
        if (try_defer(r, fd, n, off, &dret)) return dret;
    }
    if (r.flags & GSYS_F_PULL) {   // into the slot's pull area; the GPU copies it out (reading B12)
        hp = inst->pull_area(r.slot, n);
        if (!hp) return -EINVAL;
        k = PK_HOST;
    } else {
        k = resolve(buf, n, &hp);
    }
    if (k == PK_INVALID) return -EFAULT;
    if (k == PK_HOST && (r.flags & (GSYS_HOSTBUF | GSYS_F_PULL)) &&
        try_split(r, fd, hp, std::min<uint64_t>(n, GSYS_PREAD_CAP), off))   // one call returns <= the cap (A11)
        return 0;
    inst->st_host_preads.fetch_add(1, std::memory_order_relaxed);
    if (k == PK_HOST) {
        ssize_t z;
        { Timer tm(t_sys); z = pread(fd, hp, n, off); }
        if (z < 0) return -(int64_t)errno;
        inst->st_bytes_read.fetch_add((uint64_t)z, std::memory_order_relaxed);
        return z;
    }
    uint64_t want = std::min<uint64_t>(n, GSYS_PREAD_CAP);
    uint64_t piece_max = bcap / 2;
    uint64_t total = 0;
    while (total < want) {
        uint64_t piece = std::min<uint64_t>(want - total, piece_max);
        uint8_t* b = alloc(piece);
        if (!b) return total ? (int64_t)total : -ENOMEM;
        ssize_t z;
        { Timer tm(t_sys); z = pread(fd, b, piece, off + (int64_t)total); }
        if (z < 0) return total ? (int64_t)total : -(int64_t)errno;
        if (z > 0) {
            h2d((void*)(buf + total), b, (size_t)z);
            inst->st_bytes_h2d.fetch_add((uint64_t)z, std::memory_order_relaxed);
        }
        total += (uint64_t)z;
        if ((uint64_t)z < piece) break;
        if (total < want) commit();
    }
    inst->st_bytes_read.fetch_add(total, std::memory_order_relaxed);
    return (int64_t)total;
}

int64_t Worker::do_pwrite(Req& r) {
    int fd = (int)r.a[0];
    uintptr_t buf = (uintptr_t)r.a[1];
    uint64_t n = r.a[2];
    int64_t off = (int64_t)r.a[3];
    if (n == 0) {
        ssize_t z = pwrite(fd, nullptr, 0, off);
        return z < 0 ? -(int64_t)errno : 0;
    }
    uint8_t* hp = nullptr;
    PtrKind k = resolve(buf, n, &hp);
    if (k == PK_INVALID) return -EFAULT;
    if (k == PK_HOST) {
        ssize_t z = pwrite(fd, hp, n, off);
        return z < 0 ? -(int64_t)errno : z;
    }
    uint64_t want = std::min<uint64_t>(n, GSYS_PREAD_CAP);
    uint64_t piece_max = bcap / 2, total = 0;
    while (total < want) {
        uint64_t piece = std::min<uint64_t>(want - total, piece_max);
        commit();
        uint8_t* b = alloc(piece);
        if (!b) return total ? (int64_t)total : -ENOMEM;
        cudaMemcpyAsync(b, (void*)(buf + total), piece, cudaMemcpyDeviceToHost, stream);
        cudaStreamSynchronize(stream);
        ssize_t z = pwrite(fd, b, piece, off + (int64_t)total);
        if (z < 0) return total ? (int64_t)total : -(int64_t)errno;
        total += (uint64_t)z;
        if ((uint64_t)z < piece) break;
    }
    return (int64_t)total;
}

int64_t Worker::do_getrusage(Req& r) {
    struct rusage ru;
    int who = (int)(int64_t)r.a[0];
    uintptr_t dst = (uintptr_t)r.a[1];
    if (r.flags & GSYS_F_INLINE) {
        int z;
        { Timer tm(t_sys); z = getrusage(who, &ru); }
        if (z != 0) return -(int64_t)errno;
        memcpy(inst->inline_h + (size_t)r.slot * GSYS_INLINE_BYTES, &ru, sizeof ru);
        return 0;
    }
    if (dst == 0) {
        long z = syscall(SYS_getrusage, who, nullptr);
        return z < 0 ? -(int64_t)errno : 0;
    }
    if (getrusage(who, &ru) != 0) return -(int64_t)errno;
    return write_small(dst, &ru, sizeof ru);
}

// sendto / recvfrom / madvise / rt_sigqueueinfo / unknown: pointer arguments translated through
// host-mapped access or small bounce copies; then the raw syscall.
int64_t Worker::do_generic(Req& r) {
    switch (r.nr) {
        case GSYS_NR_MADVISE: {
            long z = syscall(SYS_madvise, (void*)r.a[0], (size_t)r.a[1], (int)r.a[2]);
            return z < 0 ? -(int64_t)errno : z;
        }
        case GSYS_NR_RT_SIGQUEUEINFO: {
            siginfo_t si;
            memset(&si, 0, sizeof si);
            if (r.flags & GSYS_F_INLINE_IN)
                memcpy(&si, inst->inline_h + (size_t)r.slot * GSYS_INLINE_BYTES, sizeof si);
            else if (r.a[2] && read_small((uintptr_t)r.a[2], &si, sizeof si) != 0)
                return -EFAULT;
            long z = syscall(SYS_rt_sigqueueinfo, (pid_t)r.a[0], (int)r.a[1], r.a[2] ? &si : nullptr);
            return z < 0 ? -(int64_t)errno : z;
        }
        case GSYS_NR_SENDTO: {
            size_t n = (size_t)r.a[2];
            std::vector<uint8_t> tmp(n ? n : 1);
            if (n && read_small((uintptr_t)r.a[1], tmp.data(), n) != 0) return -EFAULT;
            uint8_t sa[128];
            socklen_t salen = (socklen_t)r.a[5];
            if (r.a[4]) {
                if (salen > sizeof sa) return -EINVAL;
                if (read_small((uintptr_t)r.a[4], sa, salen) != 0) return -EFAULT;
            }
            ssize_t z = sendto((int)r.a[0], tmp.data(), n, (int)r.a[3], r.a[4] ? (struct sockaddr*)sa : nullptr,
                               r.a[4] ? salen : 0);
            return z < 0 ? -(int64_t)errno : z;
        }
        case GSYS_NR_RECVFROM:
            return do_recvfrom(r, true);
        default:
            return -ENOSYS;
    }
}

int64_t Worker::do_recvfrom(Req& r, bool may_park) {
    size_t n = (size_t)r.a[2];
    uint8_t* hp = nullptr;
    PtrKind k = resolve((uintptr_t)r.a[1], n ? n : 1, &hp);
    if (k == PK_INVALID) return -EFAULT;
    uint8_t sa[128];
    socklen_t salen = 0;
    if (r.a[5]) {
        uint32_t l = 0;
        if (read_small((uintptr_t)r.a[5], &l, 4) != 0) return -EFAULT;
        salen = std::min<uint32_t>(l, sizeof sa);
    }
    // park only calls that complete by a host store (host buffer / non-blocking) and that asked
    // to block; everything else keeps the plain blocking call
    const int uflags = (int)r.a[3];
    const bool host_done = k == PK_HOST && ((r.flags & (GSYS_HOSTBUF | GSYS_F_INLINE)) || (r.flags & GSYS_NONBLOCKING));
    const bool try_park = may_park && host_done && !(uflags & MSG_DONTWAIT);
    uint8_t* dst = hp;
    if (k == PK_DEVICE) {
        dst = alloc(n ? n : 1);
        if (!dst) return -ENOMEM;
    }
    ssize_t z = recvfrom((int)r.a[0], dst, n, uflags | (try_park || !may_park ? MSG_DONTWAIT : 0),
                         r.a[4] ? (struct sockaddr*)sa : nullptr, r.a[5] ? &salen : nullptr);
    if (z < 0) {
        const int e = errno;
        if (try_park && (e == EAGAIN || e == EWOULDBLOCK)) {
            // blocking socket? (O_NONBLOCK sockets return EAGAIN at once, as POSIX says)
            const int fl = fcntl((int)r.a[0], F_GETFL);
            if (fl >= 0 && !(fl & O_NONBLOCK)) {
                struct timeval tv = {0, 0};
                socklen_t tl = sizeof tv;
                uint64_t dl = UINT64_MAX;
                if (getsockopt((int)r.a[0], SOL_SOCKET, SO_RCVTIMEO, &tv, &tl) == 0 && (tv.tv_sec || tv.tv_usec))
                    dl = now_ns() + (uint64_t)tv.tv_sec * 1000000000ull + (uint64_t)tv.tv_usec * 1000ull;
                r.parked = true;
                std::lock_guard<std::mutex> g(inst->park_mu);
                inst->parked.push_back(Parked{r, dl});
                inst->nparked.fetch_add(1, std::memory_order_release);
                return -EAGAIN;
            }
        }
        return -(int64_t)e;
    }
    if (k == PK_DEVICE && z > 0) h2d((void*)r.a[1], dst, (size_t)z);
    if (r.a[4] && write_small((uintptr_t)r.a[4], sa, salen) != 0) return -EFAULT;
    if (r.a[5]) {
        uint32_t l = salen;
        if (write_small((uintptr_t)r.a[5], &l, 4) != 0) return -EFAULT;
    }
    return z;
}

// Retry parked recvfroms (FIFO): the first EAGAIN on a socket ends the pass for that socket;
// expired timeouts complete with -EAGAIN as the blocking call would have.
void Worker::service_parked() {
    Instance* I = inst;
    std::unique_lock<std::mutex> g(I->park_mu, std::try_to_lock);
    if (!g.owns_lock() || I->parked.empty()) return;
    const uint64_t t = now_ns();
    int empty_fd[8];
    int nempty = 0;
    size_t keep = 0;
    for (size_t i = 0; i < I->parked.size(); i++) {
        Parked p = I->parked[i];
        const int fd = (int)p.r.a[0];
        bool skip = false;
        for (int j = 0; j < nempty; j++) skip = skip || empty_fd[j] == fd;
        int64_t ret = -EAGAIN;
        bool fin = false;
        if (!skip) {
            Req r = p.r;
            r.parked = false;
            ret = do_recvfrom(r, false);
            if (ret == -EAGAIN || ret == -EWOULDBLOCK) {
                if (nempty < 8) empty_fd[nempty++] = fd;
            } else {
                fin = true;
            }
        }
        if (!fin && t >= p.deadline_ns) { fin = true; ret = -EAGAIN; }
        if (fin) {
            p.r.ret = ret;
            p.r.parked = false;
            I->complete_host(p.r);
        } else {
            I->parked[keep++] = p;
        }
    }
    const size_t done = I->parked.size() - keep;
    I->parked.resize(keep);
    if (done) I->nparked.fetch_sub((uint32_t)done, std::memory_order_release);
}

// One piece of a split pread; the worker finishing the last piece completes the request.
bool Instance::run_piece(Split& sp, uint32_t i) {
    if (i >= sp.np) return false;
    const uint64_t lo = (uint64_t)i * sp.piece;
    const uint64_t len = std::min<uint64_t>(sp.piece, sp.n - lo);
    const ssize_t z = pread(sp.fd, sp.dst + lo, len, sp.off + (int64_t)lo);
    sp.ret[i] = z < 0 ? -(int64_t)errno : (int64_t)z;
    st_host_preads.fetch_add(1, std::memory_order_relaxed);
    if (sp.done.fetch_add(1, std::memory_order_acq_rel) + 1 == sp.np) {
        int64_t total = 0;
        for (uint32_t k = 0; k < sp.np; k++) {
            const uint64_t lk = std::min<uint64_t>(sp.piece, sp.n - (uint64_t)k * sp.piece);
            if (sp.ret[k] < 0) { if (k == 0) total = sp.ret[0]; break; }
            total += sp.ret[k];
            if ((uint64_t)sp.ret[k] < lk) break;   // short piece: the single call would stop here
        }
        if (total > 0) st_bytes_read.fetch_add((uint64_t)total, std::memory_order_relaxed);
        st_split.fetch_add(1, std::memory_order_relaxed);
        sp.r.ret = total;
        complete_host(sp.r);
    }
    return true;
}

// An idle worker takes one piece of the oldest split that still has pieces left.
bool Instance::help_split() {
    std::shared_ptr<Split> sp;
    {
        std::lock_guard<std::mutex> g(split_mu);
        while (!splits.empty() && splits.front()->next.load(std::memory_order_relaxed) >= splits.front()->np) {
            splits.pop_front();
            nsplits.fetch_sub(1, std::memory_order_relaxed);
        }
        if (splits.empty()) return false;
        sp = splits.front();
    }
    return run_piece(*sp, sp->next.fetch_add(1, std::memory_order_acq_rel));
}

void Instance::complete_host(const Req& r) {
    const bool blocking = !(r.flags & GSYS_NONBLOCKING);
    gsys_slot* sl = area_h + r.slot;
    __atomic_store_n(&sl->args[0], (uint64_t)r.ret, __ATOMIC_RELAXED);
    if (r.ret < 0) {
        st_errors.fetch_add(1, std::memory_order_relaxed);
        if (!blocking) {
            int z = 0;
            first_err.compare_exchange_strong(z, (int)r.ret);
        }
    }
    if (r.ok) {
        __atomic_store_n(&sl->state, blocking ? (uint32_t)GSYS_FINISHED : (uint32_t)GSYS_FREE, __ATOMIC_RELEASE);
        host_trace(r.slot, r.seq, GSYS_PROCESSING, blocking ? GSYS_FINISHED : GSYS_FREE, blocking, r.nr);
    }
    __atomic_store_n(&hdone_h[r.slot], ((uint64_t)r.seq << 32) | (uint32_t)(int32_t)r.ret, __ATOMIC_RELEASE);
    completed.fetch_add(1, std::memory_order_release);
}

void Worker::process(uint64_t h0, uint32_t n) {
    Instance* I = inst;
    const uint64_t t_begin = now_ns();
    t_sys = t_cuda = t_wait = 0;
    const uint32_t mask = I->ring_cap - 1;
    reqs.resize(n);
    for (uint32_t i = 0; i < n; i++) {
        uint64_t e = __atomic_load_n(&I->ring_h[(h0 + i) & mask], __ATOMIC_ACQUIRE);
        Req& r = reqs[i];
        r.slot = (uint32_t)e;
        r.pos = (uint32_t)(h0 + i);
        // the line was written by the GPU before its doorbell entry (fence.acq_rel.sys + the entry
        // load above); plain atomic loads, since another worker may still be storing args[0] of the
        // slot's previous request (ordered only through the GPU, which the C++ model cannot see)
        gsys_slot* sl = I->area_h + r.slot;
        r.nr = __atomic_load_n(&sl->nr, __ATOMIC_RELAXED);
        r.flags = __atomic_load_n(&sl->flags, __ATOMIC_RELAXED);
        r.seq = __atomic_load_n(&sl->seq, __ATOMIC_RELAXED);
        for (int k = 0; k < 6; k++) r.a[k] = __atomic_load_n(&sl->args[k], __ATOMIC_RELAXED);
        r.ret = 0;
        r.dma = false;
        r.parked = false;
        r.faulted = false;
        r.early = false;
        r.dropped = false;
        // "atomically switches any ready system call requests to the processing state" (P24.20)
        uint32_t expect = GSYS_READY;
        r.ok = __atomic_compare_exchange_n((uint32_t*)&I->area_h[r.slot].state, &expect, (uint32_t)GSYS_PROCESSING,
                                           false, __ATOMIC_ACQ_REL, __ATOMIC_ACQUIRE);
        if (!r.ok) r.ret = -EPROTO;
        else I->host_trace(r.slot, r.seq, GSYS_READY, GSYS_PROCESSING, !(r.flags & GSYS_NONBLOCKING), r.nr);
        I->st_nr[nr_index(r.nr)].fetch_add(1, std::memory_order_relaxed);
    }

    // ---- fault injection (tests): the pread at the chosen offset fails without being executed
    std::vector<uint8_t>& done = done_;   // reused per bundle (no allocation per request)
    done.assign(n, 0);
    if (const int ferr = I->fault_err.load(std::memory_order_relaxed)) {
        const int64_t foff = I->fault_off.load(std::memory_order_relaxed);
        for (uint32_t i = 0; i < n; i++) {
            Req& r = reqs[i];
            if (r.ok && r.nr == GSYS_NR_PREAD64 && (int64_t)r.a[3] == foff) {
                r.ret = -(int64_t)ferr;
                r.faulted = true;
                done[i] = true;
                I->st_faults.fetch_add(1, std::memory_order_relaxed);
            }
        }
    }
    if (I->drop_off.load(std::memory_order_relaxed) >= 0) {
        const int64_t doff = I->drop_off.load(std::memory_order_relaxed);
        for (uint32_t i = 0; i < n; i++) {
            Req& r = reqs[i];
            if (r.ok && r.nr == GSYS_NR_PREAD64 && (int64_t)r.a[3] == doff) {
                r.dropped = true;
                I->st_faults.fetch_add(1, std::memory_order_relaxed);
            }
        }
    }
    // ---- execute: preads first through the merge planner (reading A8), then the rest in order
    midx.clear();
    for (uint32_t i = 0; i < n; i++)
        if (reqs[i].ok && reqs[i].nr == GSYS_NR_PREAD64 && !reqs[i].faulted) midx.push_back(i);
    if (midx.size() > 1 && I->merge.load(std::memory_order_relaxed)) {
        uint32_t m = (uint32_t)midx.size();
        mfd.resize(m); moff.resize(m); mlen.resize(m); morder.resize(m); mgroup.resize(m);
        mgoff_in.resize(m); mg_off.resize(m); mg_len.resize(m);
        for (uint32_t j = 0; j < m; j++) {
            Req& r = reqs[midx[j]];
            mfd[j] = (int32_t)r.a[0]; moff[j] = (int64_t)r.a[3]; mlen[j] = r.a[2];
        }
        int ng = gsys_plan_merge(m, mfd.data(), moff.data(), mlen.data(), bcap / 2, morder.data(), mgroup.data(),
                                 mgoff_in.data(), mg_off.data(), mg_len.data());
        // execute groups with >= 2 members on regular files whose destinations are all resolvable
        std::vector<std::vector<uint32_t>>& members = members_;
        if (members.size() < (size_t)(ng > 0 ? ng : 0)) members.resize(ng);
        for (int g = 0; g < ng; g++) members[g].clear();
        for (uint32_t t = 0; t < m; t++) members[mgroup[morder[t]]].push_back(morder[t]);
        for (int g = 0; g < ng; g++) {
            auto& mem = members[g];
            if (mem.size() < 2) continue;
            int fd = mfd[mem[0]];
            struct stat st;
            if (fstat(fd, &st) != 0 || !S_ISREG(st.st_mode)) continue;
            // merge only where it saves work: device destinations go through the bounce anyway;
            // for large reads into host memory the union read would add a second memcpy
            bool okd = true;
            for (uint32_t j : mem) {
                Req& r = reqs[midx[j]];
                // read alone into the bounce (B13) / a deferred range (B15): a merged read would land
                // by DMA, out of order with the deferred pulls
                if (r.flags & (GSYS_F_PULLB | GSYS_F_DEFER)) { okd = false; break; }
                PtrKind k = !r.a[2] ? PK_INVALID
                            : (r.flags & GSYS_F_PULL) ? (I->pull_area(r.slot, r.a[2]) ? PK_HOST : PK_INVALID)
                                                      : resolve((uintptr_t)r.a[1], r.a[2], nullptr);
                if (k == PK_INVALID || (k == PK_HOST && r.a[2] > (64u << 10))) { okd = false; break; }
            }
            if (!okd) continue;
            uint8_t* b = alloc(mg_len[g]);
            if (!b) continue;
            ssize_t z;
            { Timer tm(t_sys); z = pread(fd, b, mg_len[g], mg_off[g]); }
            I->st_host_preads.fetch_add(1, std::memory_order_relaxed);
            int64_t zr = z < 0 ? -(int64_t)errno : (int64_t)z;
            if (zr > 0) I->st_bytes_read.fetch_add((uint64_t)zr, std::memory_order_relaxed);
            for (uint32_t j : mem) {
                Req& r = reqs[midx[j]];
                int64_t ri = gsys_split_result(zr, mgoff_in[j], r.a[2]);
                r.ret = ri;
                done[midx[j]] = true;
                dma_flag = false;
                if (ri > 0) {
                    uint8_t* hp = nullptr;
                    PtrKind k = PK_HOST;
                    if (r.flags & GSYS_F_PULL) hp = I->pull_area(r.slot, r.a[2]);
                    else k = resolve((uintptr_t)r.a[1], r.a[2], &hp);
                    if (k == PK_HOST) {
                        memcpy(hp, b + mgoff_in[j], (size_t)ri);
                    } else {
                        h2d((void*)r.a[1], b + mgoff_in[j], (size_t)ri);
                        I->st_bytes_h2d.fetch_add((uint64_t)ri, std::memory_order_relaxed);
                    }
                }
                r.dma = dma_flag;
            }
            I->st_merged.fetch_add(mem.size(), std::memory_order_relaxed);
        }
        // remaining preads in (fd, off) order
        for (uint32_t t = 0; t < m; t++) {
            uint32_t i = midx[morder[t]];
            if (done[i]) continue;
            dma_flag = false;
            reqs[i].ret = do_pread(reqs[i]);
            reqs[i].dma = dma_flag;
            done[i] = true;
        }
    }
    for (uint32_t i = 0; i < n; i++) {
        Req& r = reqs[i];
        if (!r.ok || done[i]) continue;
        dma_flag = false;
        switch (r.nr) {
            case GSYS_NR_PREAD64: r.ret = do_pread(r); break;
            case GSYS_NR_PWRITE64: r.ret = do_pwrite(r); break;
            case GSYS_NR_GETRUSAGE: r.ret = do_getrusage(r); break;
            default: r.ret = do_generic(r); break;
        }
        r.dma = dma_flag;
    }

    flush_copies();
    // ---- completion (P24.32-35): result into args[0]; blocking -> "finished" + completion word,
    // non-blocking -> "free" + completion word (which the slot's next GPU claimer waits for).
    // Non-blocking, GSYS_HOSTBUF and inline requests complete with a host store into the
    // host-mapped word (after their DMA, if any, has drained); blocking requests for device
    // buffers complete with a stream memory operation ordered after the DMA above.
    ops.clear();
    bool need_sync = false;
    uint32_t nparked_here = 0;   // parked or already completed: not counted below
    for (uint32_t i = 0; i < n; i++) {
        Req& r = reqs[i];
        if (r.parked || r.early) { nparked_here++; continue; }
        if (r.dropped) continue;   // fault injection: drained, the completion is never written
        const bool blocking = !(r.flags & GSYS_NONBLOCKING);
        gsys_slot* sl = I->area_h + r.slot;
        __atomic_store_n(&sl->args[0], (uint64_t)r.ret, __ATOMIC_RELAXED);
        if (r.ret < 0) {
            I->st_errors.fetch_add(1, std::memory_order_relaxed);
            if (!blocking) {
                int z = 0;
                I->first_err.compare_exchange_strong(z, (int)r.ret);
            }
        }
        CUstreamBatchMemOpParams op;
        memset(&op, 0, sizeof op);
        if (blocking) {
            const uint64_t word = ((uint64_t)r.seq << 32) | (uint32_t)(int32_t)r.ret;
            if (!I->memop_completion || (r.flags & (GSYS_HOSTBUF | GSYS_F_INLINE | GSYS_F_PULL))) {
                if (r.dma) { need_sync = true; continue; }
                if (r.ok) {
                    __atomic_store_n(&sl->state, (uint32_t)GSYS_FINISHED, __ATOMIC_RELEASE);
                    I->host_trace(r.slot, r.seq, GSYS_PROCESSING, GSYS_FINISHED, true, r.nr);
                }
                __atomic_store_n(&I->hdone_h[r.slot], word, __ATOMIC_RELEASE);
                continue;
            }
            if (r.ok) {
                __atomic_store_n(&sl->state, (uint32_t)GSYS_FINISHED, __ATOMIC_RELEASE);
                I->host_trace(r.slot, r.seq, GSYS_PROCESSING, GSYS_FINISHED, true, r.nr);
            }
            if (I->mem64) {
                op.writeValue.operation = CU_STREAM_MEM_OP_WRITE_VALUE_64;
                op.writeValue.address = (CUdeviceptr)(I->mirror_d + r.slot);
                op.writeValue.value64 = word;
                op.writeValue.flags = CU_STREAM_WRITE_VALUE_DEFAULT;
                ops.push_back(op);
            } else {
                op.writeValue.operation = CU_STREAM_MEM_OP_WRITE_VALUE_32;
                op.writeValue.address = (CUdeviceptr)(I->mirror_d + r.slot);
                op.writeValue.value = (uint32_t)word;
                op.writeValue.flags = CU_STREAM_WRITE_VALUE_DEFAULT;
                ops.push_back(op);
                op.writeValue.address = (CUdeviceptr)((uint8_t*)(I->mirror_d + r.slot) + 4);
                op.writeValue.value = (uint32_t)(word >> 32);
                ops.push_back(op);
            }
        } else {
            // non-blocking: "the state is changed to free" (P24.34); the GPU's next claimer of this
            // slot waits for the host-mapped completion word (after any DMA has drained)
            if (r.dma) { need_sync = true; continue; }
            if (r.ok) {
                __atomic_store_n(&sl->state, (uint32_t)GSYS_FREE, __ATOMIC_RELEASE);
                I->host_trace(r.slot, r.seq, GSYS_PROCESSING, GSYS_FREE, false, r.nr);
            }
            __atomic_store_n(&I->hdone_h[r.slot], ((uint64_t)r.seq << 32) | (uint32_t)(int32_t)r.ret,
                             __ATOMIC_RELEASE);
        }
    }
    if (need_sync) {
        // host-store completions whose payload went through the DMA: wait for it to land first
        cudaEvent_t e = get_event();
        {
            Timer tm(t_wait);
            cudaEventRecord(e, stream);
            cudaEventSynchronize(e);
        }
        evpool.push_back(e);
        for (uint32_t i = 0; i < n; i++) {
            Req& r = reqs[i];
            const bool nb = (r.flags & GSYS_NONBLOCKING) != 0;
            if (r.dropped || r.early || r.parked) continue;
            if (!r.dma || (!nb && I->memop_completion && !(r.flags & (GSYS_HOSTBUF | GSYS_F_INLINE | GSYS_F_PULL))))
                continue;
            gsys_slot* sl = I->area_h + r.slot;
            if (r.ok) {
                __atomic_store_n(&sl->state, nb ? (uint32_t)GSYS_FREE : (uint32_t)GSYS_FINISHED, __ATOMIC_RELEASE);
                I->host_trace(r.slot, r.seq, GSYS_PROCESSING, nb ? GSYS_FREE : GSYS_FINISHED, !nb, r.nr);
            }
            __atomic_store_n(&I->hdone_h[r.slot], ((uint64_t)r.seq << 32) | (uint32_t)(int32_t)r.ret,
                             __ATOMIC_RELEASE);
        }
    }
    for (size_t i = 0; i < ops.size(); i += 128) {
        unsigned cnt = (unsigned)std::min<size_t>(128, ops.size() - i);
        CUresult cr;
        { Timer tm(t_cuda); cr = p_batch((CUstream)stream, cnt, ops.data() + i, 0); }
        if (cr != CUDA_SUCCESS) {
            fprintf(stderr, "gsys: cuStreamBatchMemOp failed (%d)\n", (int)cr);
            int z = 0;
            I->first_err.compare_exchange_strong(z, -EIO);
        }
    }
    commit();
    I->completed.fetch_add(n - nparked_here, std::memory_order_release);
    I->st_ns_busy.fetch_add(now_ns() - t_begin, std::memory_order_relaxed);
    I->st_ns_syscall.fetch_add(t_sys, std::memory_order_relaxed);
    I->st_ns_cuda.fetch_add(t_cuda, std::memory_order_relaxed);
    I->st_ns_wait.fetch_add(t_wait, std::memory_order_relaxed);
}

int make_instance(uint32_t slots, uint32_t window_us, Instance** out) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return -ENODEV;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) return -ENODEV;
    cudaFree(0);   // make the primary context current
    if (!p_batch) {
        cudaDriverEntryPointQueryResult q;
        void* fn = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamBatchMemOp", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn)
            return -ENOTSUP;
        p_batch = (PFN_batch_t)fn;
        fn = nullptr;
        if (cudaGetDriverEntryPoint("cuPointerGetAttributes", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn)
            return -ENOTSUP;
        p_ptrattrs = (PFN_ptrattrs_t)fn;
        fn = nullptr;
        if (cudaGetDriverEntryPoint("cuDeviceGetAttribute", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn)
            return -ENOTSUP;
        p_devattr = (PFN_devattr_t)fn;
        fn = nullptr;
        if (cudaGetDriverEntryPoint("cuLaunchKernel", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn)
            return -ENOTSUP;
        p_launch = (PFN_launch_t)fn;
        fn = nullptr;
        if (cudaGetDriverEntryPoint("cuFuncSetAttribute", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn)
            return -ENOTSUP;
        p_funcsetattr = (PFN_funcsetattr_t)fn;
    }
    Instance* I = new Instance();
    I->dev = dev;
    int v = 0;
    I->mem64 = (p_devattr(&v, CU_DEVICE_ATTRIBUTE_CAN_USE_64_BIT_STREAM_MEM_OPS, dev) == CUDA_SUCCESS && v);
    int sms = 0, thr_per_sm = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaDeviceGetAttribute(&thr_per_sm, cudaDevAttrMaxThreadsPerMultiProcessor, dev);
    if (slots == 0) {
        // %smid may exceed the SM count on partially-enabled dies: size for 2x headroom, the
        // hardware-ID hash (modulo) + claim CAS keep it correct for any value (reading A5).
        uint64_t s = (uint64_t)sms * 2048ull;
        slots = (uint32_t)std::min<uint64_t>(s, 1u << 24);
    }
    I->nslots = slots;
    uint32_t rc = 1;
    while (rc < slots + 1024u) rc <<= 1;
    I->ring_cap = rc;
    I->window_us.store(window_us);
    const char* ev = getenv("GSYS_COALESCE_MAX");
    if (ev && atoi(ev) > 0) I->coalesce_max.store((uint32_t)atoi(ev));
    ev = getenv("GSYS_MERGE");
    if (ev) I->merge.store(atoi(ev) ? 1 : 0);

    auto fail = [&](int code) { /* leak on failure paths: rare, process-lifetime */ delete I; return code; };
    size_t area_bytes = (size_t)slots * sizeof(gsys_slot);
    if (cudaHostAlloc((void**)&I->area_h, area_bytes, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
        return fail(-ENOMEM);
    memset(I->area_h, 0, area_bytes);
    if (cudaHostGetDevicePointer((void**)&I->area_d, I->area_h, 0) != cudaSuccess) return fail(-EIO);
    size_t inl = (size_t)slots * GSYS_INLINE_BYTES;
    if (cudaHostAlloc((void**)&I->inline_h, inl, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
        return fail(-ENOMEM);
    if (cudaHostGetDevicePointer((void**)&I->inline_d, I->inline_h, 0) != cudaSuccess) return fail(-EIO);
    {   // pull areas of the slots a work-group caller lands in (s % 32 == 0): GSYS_PULL_KB, default 16
        const char* pv = getenv("GSYS_PULL_KB");
        const long kb = pv ? atol(pv) : 16;
        I->pull_bytes = (kb > 0 && kb <= 1024) ? (uint32_t)kb << 10 : 0u;
        const size_t pb = (size_t)((slots + 31) / 32) * I->pull_bytes;
        if (pb && cudaHostAlloc((void**)&I->pull_h, pb, cudaHostAllocMapped | cudaHostAllocPortable) == cudaSuccess) {
            if (cudaHostGetDevicePointer((void**)&I->pull_d, I->pull_h, 0) != cudaSuccess) return fail(-EIO);
        } else {
            cudaGetLastError();
            I->pull_h = nullptr;
            I->pull_bytes = 0;
        }
    }
    if (cudaHostAlloc((void**)&I->ring_h, (size_t)rc * 8, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
        return fail(-ENOMEM);
    memset(I->ring_h, 0, (size_t)rc * 8);
    if (cudaHostGetDevicePointer((void**)&I->ring_d, I->ring_h, 0) != cudaSuccess) return fail(-EIO);
    // deferred-pull records, one per ring position (B15)
    if (cudaHostAlloc((void**)&I->nbrec_h, (size_t)rc * sizeof(gsys_nbrec), cudaHostAllocMapped | cudaHostAllocPortable) !=
        cudaSuccess)
        return fail(-ENOMEM);
    memset(I->nbrec_h, 0, (size_t)rc * sizeof(gsys_nbrec));
    if (cudaHostGetDevicePointer((void**)&I->nbrec_d, I->nbrec_h, 0) != cudaSuccess) return fail(-EIO);
    if (cudaHostAlloc((void**)&I->hdone_h, (size_t)slots * 8, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
        return fail(-ENOMEM);
    memset(I->hdone_h, 0, (size_t)slots * 8);
    if (cudaHostGetDevicePointer((void**)&I->hdone_d, I->hdone_h, 0) != cudaSuccess) return fail(-EIO);
    if (cudaMalloc(&I->claim_d, (size_t)slots * 4) != cudaSuccess) return fail(-ENOMEM);
    if (cudaMalloc(&I->seqs_d, (size_t)slots * 4) != cudaSuccess) return fail(-ENOMEM);
    if (cudaMalloc(&I->mirror_d, (size_t)slots * 8) != cudaSuccess) return fail(-ENOMEM);
    if (cudaMalloc(&I->tail_d, 64) != cudaSuccess) return fail(-ENOMEM);
    if (cudaMalloc(&I->lat_hint_d, (size_t)slots * 4) != cudaSuccess) return fail(-ENOMEM);
    cudaMemset(I->lat_hint_d, 0, (size_t)slots * 4);
    if (cudaMalloc(&I->nbpend_d, (size_t)slots * 4) != cudaSuccess) return fail(-ENOMEM);
    cudaMemset(I->nbpend_d, 0, (size_t)slots * 4);
    if (cudaMalloc(&I->nbpos_d, (size_t)slots * 4) != cudaSuccess) return fail(-ENOMEM);
    cudaMemset(I->nbpos_d, 0, (size_t)slots * 4);
    if (cudaMalloc(&I->nbclaim_d, (size_t)rc * 4) != cudaSuccess) return fail(-ENOMEM);
    cudaMemset(I->nbclaim_d, 0, (size_t)rc * 4);
    if (cudaMalloc(&I->krounds_d, sizeof(gsys_kround) * GSYS_KSITES * GSYS_KROUNDS) != cudaSuccess) return fail(-ENOMEM);
    I->kblock_cap = 4096;
    if (cudaMalloc(&I->kblock_d, (size_t)I->kblock_cap * GSYS_KSITES * 4) != cudaSuccess) return fail(-ENOMEM);
    cudaMemset(I->claim_d, 0, (size_t)slots * 4);
    cudaMemset(I->seqs_d, 0, (size_t)slots * 4);
    cudaMemset(I->mirror_d, 0, (size_t)slots * 8);
    cudaMemset(I->tail_d, 0, 64);
    cudaMemset(I->krounds_d, 0, sizeof(gsys_kround) * GSYS_KSITES * GSYS_KROUNDS);
    cudaMemset(I->kblock_d, 0, (size_t)I->kblock_cap * GSYS_KSITES * 4);
    if (cudaMalloc(&I->ctx_d, sizeof(gsys_dev_ctx)) != cudaSuccess) return fail(-ENOMEM);
    if (cudaStreamCreateWithFlags(&I->ctl, cudaStreamNonBlocking) != cudaSuccess) return fail(-EIO);
    gsys_dev_ctx& c = I->ctx_h;
    c.area = I->area_d;
    c.inline_buf = I->inline_d;
    c.claim = I->claim_d;
    c.seqs = I->seqs_d;
    c.mirror = I->mirror_d;
    c.hdone = (unsigned long long*)I->hdone_d;
    c.lat_hint = I->lat_hint_d;
    c.nbpend = I->nbpend_d;
    c.nbpos = I->nbpos_d;
    c.nbclaim = I->nbclaim_d;
    c.ring = (unsigned long long*)I->ring_d;
    c.ring_tail = I->tail_d;
    c.krounds = I->krounds_d;
    c.kblock = I->kblock_d;
    c.kblock_cap = I->kblock_cap;
    c.trace = nullptr;
    c.trace_n = nullptr;
    c.trace_cap = 0;
    c.nslots = slots;
    c.ring_mask = rc - 1;
    ev = getenv("GSYS_POLL_NS_MAX");
    c.poll_ns_max = (ev && atoi(ev) > 0) ? (unsigned)atoi(ev) : 1024u;
    ev = getenv("GSYS_POLL_NS_HOST");
    // 256 ns: a 4 KiB pread round trip drops from 16.1 to 9.9 us vs 4 us polling, and the
    // wordcount (pollers sharing the PCIe link with the scan) is unchanged (profiles/r01_latency.json)
    c.poll_ns_host = (ev && atoi(ev) > 0) ? (unsigned)atoi(ev) : 256u;
    // completion path of blocking device-buffer calls (gsys.h GSYS_COMPLETION_*), env
    // GSYS_COMPLETION=memop|host|pull.  Default pull (reading B13): the work-group copies its bytes
    // out of the service's host-mapped bounce -- 8 GiB device-staged wordcount 50.5 GB/s vs 24.5
    // (memop) / 23.6 (host), WG 64 KiB device preads 0.75 M/s vs 0.09 / 0.14 M/s
    // (profiles/r02_completion_ab.jsonl); the copy-engine paths pay CUDA API calls per request.
    ev = getenv("GSYS_COMPLETION");
    const int cmode = !ev ? 2 : strcmp(ev, "memop") == 0 ? 0 : strcmp(ev, "host") == 0 ? 1 : 2;
    c.memop_completion = cmode == 0 ? 1u : 0u;
    c.pull_bounce = cmode == 2 ? 1u : 0u;
    I->memop_completion = c.memop_completion != 0;
    ev = getenv("GSYS_BIG_ALONE");
    I->big_alone = !(ev && atoi(ev) == 0);
    ev = getenv("GSYS_SPLIT_KB");
    if (ev) I->split_min = (uint64_t)atoll(ev) << 10;
    ev = getenv("GSYS_SHARE_BURSTS");
    I->share_bursts = !(ev && atoi(ev) == 0);
    ev = getenv("GSYS_DIAG_PHASES");
    if (ev && atoi(ev) > 0) {
        if (cudaMalloc((void**)&c.diag, 64) != cudaSuccess) return fail(-ENOMEM);
        cudaMemset(c.diag, 0, 64);
        I->diag_d = c.diag;
    }
    ev = getenv("GSYS_SLEEP_HINT");
    c.no_hint = (ev && atoi(ev) == 0) ? 1u : 0u;
    // watchdog: GSYS_POLL_TIMEOUT_MS, default 20 s, 0 = off
    ev = getenv("GSYS_POLL_TIMEOUT_MS");
    c.poll_timeout_ns = (unsigned long long)(ev ? atoll(ev) : 20000ll) * 1000000ull;
    if (cudaMalloc((void**)&I->wd_d, sizeof(gsys_wd_log)) != cudaSuccess) return fail(-ENOMEM);
    cudaMemset(I->wd_d, 0, sizeof(gsys_wd_log));
    c.wd = I->wd_d;
    ev = getenv("GSYS_DEFER_MB");   // per worker; 0 = non-blocking device-buffer preads by DMA
    const size_t defer_mb = ev ? (size_t)atoll(ev) : 16;
    ev = getenv("GSYS_DEFER_GROW_MB");
    I->defer_grow = (size_t)(ev ? atoll(ev) : 64) << 20;
    c.nbrec = defer_mb ? (gsys_nbrec*)I->nbrec_d : nullptr;
    c.pull_big_bytes = I->pull_bytes;
    c.pull_big = I->pull_d;
    if (cudaMemcpy(I->ctx_d, &c, sizeof c, cudaMemcpyHostToDevice) != cudaSuccess) return fail(-EIO);
    if (preload_flush_kernel() != 0) return fail(-EIO);
    if (cudaDeviceSynchronize() != cudaSuccess) return fail(-EIO);

    // service threads: on the CPUs local to this GPU's PCIe root, sized for the
    // ranks that share the host (LOCAL_WORLD_SIZE, set by torchrun)
    const int nlocal = service_cpus(I->dev, &I->cpus);
    uint32_t nthr;
    {
        const char* lw = getenv("LOCAL_WORLD_SIZE");
        const long lws = (lw && atol(lw) > 0) ? atol(lw) : 1;
        long allowed = (long)std::thread::hardware_concurrency();
        cpu_set_t cs;
        if (sched_getaffinity(0, sizeof cs, &cs) == 0) allowed = CPU_COUNT(&cs);
        // ranks expected on this GPU's CPU set if the GPUs are spread evenly across NUMA nodes
        const long share = std::max<long>(1, (lws * nlocal + allowed - 1) / std::max<long>(1, allowed));
        const long per = nlocal / share;
        nthr = (uint32_t)std::max<long>(1, std::min<long>(16, lws == 1 ? per - 2 : per - 1));
    }
    ev = getenv("GSYS_THREADS");
    if (ev && atoi(ev) > 0) nthr = (uint32_t)atoi(ev);
    I->nthreads = nthr;
    size_t bcap = 32ull << 20;
    ev = getenv("GSYS_BOUNCE_MB");
    if (ev && atoi(ev) > 0) bcap = (size_t)atoi(ev) << 20;
    for (uint32_t t = 0; t < nthr; t++) {
        Worker* w = new Worker();
        w->inst = I;
        w->id = (int)t;
        if (cudaStreamCreateWithFlags(&w->stream, cudaStreamNonBlocking) != cudaSuccess) { delete w; return fail(-EIO); }
        if (cudaHostAlloc((void**)&w->bounce, bcap, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) {
            delete w;
            return fail(-ENOMEM);
        }
        if (cudaHostGetDevicePointer((void**)&w->bounce_d, w->bounce, 0) != cudaSuccess) { delete w; return fail(-EIO); }
        if (defer_mb) {
            w->defer.cap = defer_mb << 20;
            if (cudaHostAlloc((void**)&w->defer.h, w->defer.cap, cudaHostAllocMapped | cudaHostAllocPortable) !=
                    cudaSuccess ||
                cudaHostGetDevicePointer((void**)&w->defer.d, w->defer.h, 0) != cudaSuccess) {
                delete w;
                return fail(-ENOMEM);
            }
            w->defer.recs = I->nbrec_h;
            w->defer.mask = rc - 1;
        }
        w->bcap = bcap;
        w->ring = new BounceRing<Worker::Tok, Worker::RingOps>(bcap, &w->ring_ops);
        w->reqs.reserve(4096);
        w->ops.reserve(8192);
        I->workers.push_back(w);
    }
    for (Worker* w : I->workers) w->th = std::thread([w] { w->run(); });
    *out = I;
    return 0;
}

}  // namespace

// ====================================================================== internal API
gsys_dev_ctx* gsys_internal_ctx_d() {
    Instance* I = current();
    return I ? I->ctx_d : nullptr;
}
void gsys_internal_register_host_range(const void* p, size_t n, int add) {
    const uintptr_t lo = (uintptr_t)p, hi = lo + n;
    if (add) {
        int i = g_nhost_ranges.load();
        if (i >= 32) return;
        g_host_ranges[i].lo.store(lo);
        g_host_ranges[i].hi.store(hi);
        g_nhost_ranges.store(i + 1, std::memory_order_release);
    } else {
        // ranges are only removed when the library frees them, i.e. while no call can use them
        int nr = g_nhost_ranges.load();
        for (int i = 0; i < nr; i++)
            if (g_host_ranges[i].lo.load() == lo) { g_host_ranges[i].lo.store(1); g_host_ranges[i].hi.store(0); }
    }
}

int gsys_internal_nslots() {
    Instance* I = current();
    return I ? (int)I->nslots : 0;
}

// ====================================================================== C-ABI
extern "C" {

int gsys_init(uint32_t slots, uint32_t coalesce_window_us) {
    if (slots > (1u << 24)) return -EINVAL;
    std::lock_guard<std::mutex> g(g_mu);
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess) return -ENODEV;
    if (d < 0 || d >= 64) return -ENODEV;
    if (g_inst[d]) return -EALREADY;
    Instance* I = nullptr;
    int r = make_instance(slots, coalesce_window_us, &I);
    if (r) return r;
    g_inst[d] = I;
    return 0;
}

int gsys_set_coalesce_max(uint32_t n) {
    if (n == 0 || n > 4096) return -EINVAL;
    Instance* I = current();
    if (!I) return -ENODEV;
    I->coalesce_max.store(n);
    return 0;
}

int gsys_set_coalesce_window(uint32_t us) {
    Instance* I = current();
    if (!I) return -ENODEV;
    I->window_us.store(us);
    return 0;
}

int gsys_diag_phases(uint64_t* out8, int reset) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (!I->diag_d) return -ENOTSUP;
    if (!out8) return -EINVAL;
    if (cudaMemcpy(out8, I->diag_d, 64, cudaMemcpyDeviceToHost) != cudaSuccess) return -EIO;
    if (reset && cudaMemset(I->diag_d, 0, 64) != cudaSuccess) return -EIO;
    return 0;
}

int gsys_set_fault(int32_t err, int64_t offset) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (err < 0 || err > 4095) return -EINVAL;
    I->fault_off.store(offset);
    I->fault_err.store(err);
    return 0;
}

int gsys_set_merge(int on) {
    Instance* I = current();
    if (!I) return -ENODEV;
    I->merge.store(on ? 1 : 0);
    return 0;
}

int gsys_set_trace(int on, uint32_t capacity) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (gsys_wait(nullptr) < -1000) return -EIO;
    if (on) {
        if (capacity == 0) capacity = 1u << 20;
        if (I->gtrace_d) { I->graveyard.push_back(I->gtrace_d); I->graveyard.push_back(I->gtrace_n_d); }
        if (cudaMalloc(&I->gtrace_d, (size_t)capacity * sizeof(gsys_trace_rec)) != cudaSuccess) return -ENOMEM;
        if (cudaMalloc(&I->gtrace_n_d, 64) != cudaSuccess) return -ENOMEM;
        cudaMemset(I->gtrace_n_d, 0, 64);
        I->trace_cap = capacity;
        {
            std::lock_guard<std::mutex> g(I->trace_mu);
            I->htrace.clear();
            I->htrace.reserve(capacity);
        }
        I->ctx_h.trace = I->gtrace_d;
        I->ctx_h.trace_n = I->gtrace_n_d;
        I->ctx_h.trace_cap = capacity;
        I->tracing.store(1);
    } else {
        I->tracing.store(0);
        I->ctx_h.trace = nullptr;
        I->ctx_h.trace_n = nullptr;
        I->ctx_h.trace_cap = 0;
    }
    if (cudaMemcpy(I->ctx_d, &I->ctx_h, sizeof I->ctx_h, cudaMemcpyHostToDevice) != cudaSuccess) return -EIO;
    return 0;
}

int gsys_trace_read(gsys_trace_rec* gpu_out, uint32_t gpu_cap, uint32_t* n_gpu, gsys_trace_rec* host_out,
                    uint32_t host_cap, uint32_t* n_host) {
    Instance* I = current();
    if (!I) return -ENODEV;
    uint32_t ng = 0;
    if (I->gtrace_n_d) {
        cudaMemcpy(&ng, I->gtrace_n_d, 4, cudaMemcpyDeviceToHost);
        ng = std::min(ng, I->trace_cap);
        uint32_t k = std::min(ng, gpu_cap);
        if (k && gpu_out) cudaMemcpy(gpu_out, I->gtrace_d, (size_t)k * sizeof(gsys_trace_rec), cudaMemcpyDeviceToHost);
        cudaMemset(I->gtrace_n_d, 0, 4);
    }
    if (n_gpu) *n_gpu = ng;
    std::lock_guard<std::mutex> g(I->trace_mu);
    uint32_t nh = (uint32_t)I->htrace.size();
    uint32_t k = std::min(nh, host_cap);
    if (k && host_out) memcpy(host_out, I->htrace.data(), (size_t)k * sizeof(gsys_trace_rec));
    if (n_host) *n_host = nh;
    I->htrace.clear();
    return 0;
}

}  // extern "C"
static int launch_begin_impl(uint64_t nblocks, void* stream, bool ksites) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (nblocks == 0 || nblocks > (1ull << 31)) return -EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    const uint64_t nb = nblocks;
    if (nb > I->kblock_cap) {
        uint32_t cap = I->kblock_cap;
        while (cap < nb) cap <<= 1;
        uint32_t* nk = nullptr;
        if (cudaMalloc(&nk, (size_t)cap * GSYS_KSITES * 4) != cudaSuccess) return -ENOMEM;
        cudaDeviceSynchronize();   // no running kernel may still read the old array
        I->graveyard.push_back(I->kblock_d);
        I->kblock_d = nk;
        I->kblock_cap = cap;
        I->ctx_h.kblock = nk;
        I->ctx_h.kblock_cap = cap;
        if (cudaMemcpy(I->ctx_d, &I->ctx_h, sizeof I->ctx_h, cudaMemcpyHostToDevice) != cudaSuccess) return -EIO;
    }
    // reset the kernel-scope call sites for this launch (block rounds + per-round records); they
    // are shared by the instance: kernel-scope calls of launches running concurrently on other
    // streams are not supported (gsys.h).  Library kernels that make no kernel-scope call skip it.
    if (ksites) {
        cudaMemsetAsync(I->kblock_d, 0, (size_t)nb * GSYS_KSITES * 4, s);
        cudaMemsetAsync(I->krounds_d, 0, sizeof(gsys_kround) * GSYS_KSITES * GSYS_KROUNDS, s);
    }
    // the learned pre-poll sleep (reading B3) is relearned per launch: a hint carried over from
    // another workload's latency would make this kernel's first calls oversleep
    cudaMemsetAsync(I->lat_hint_d, 0, (size_t)I->nslots * 4, s);
    I->gen.fetch_add(1);
    I->kick.fetch_add(1);
    if (I->sleepers.load(std::memory_order_relaxed) > 0) {
        std::lock_guard<std::mutex> lk(I->sleep_mu);
        I->sleep_cv.notify_all();
    }
    return cuda_err(cudaGetLastError());
}

int gsys_internal_launch(const void* kernel, uint32_t grid, uint32_t block, void** args, size_t smem, void* stream,
                         bool kernel_sites) {
    if (!kernel || grid == 0 || block == 0) return -EINVAL;
    int rc = launch_begin_impl(grid, stream, kernel_sites);
    if (rc) return rc;
    return cuda_err(cudaLaunchKernel(kernel, dim3(grid), dim3(block), args, smem, (cudaStream_t)stream));
}

extern "C" {

int gsys_launch_begin(uint64_t nblocks, void* stream) { return launch_begin_impl(nblocks, stream, true); }

int gsys_launch(const void* kernel, uint32_t gx, uint32_t gy, uint32_t gz, uint32_t bx, uint32_t by, uint32_t bz,
                void** args, size_t smem_bytes, void* stream) {
    if (!kernel || gx == 0 || gy == 0 || gz == 0 || bx == 0 || by == 0 || bz == 0) return -EINVAL;
    int rc = gsys_launch_begin((uint64_t)gx * gy * gz, stream);
    if (rc) return rc;
    return cuda_err(cudaLaunchKernel(kernel, dim3(gx, gy, gz), dim3(bx, by, bz), args, smem_bytes,
                                     (cudaStream_t)stream));
}

int gsys_launch_cu(void* cu_function, uint32_t gx, uint32_t gy, uint32_t gz, uint32_t bx, uint32_t by, uint32_t bz,
                   void** args, size_t smem_bytes, void* stream) {
    if (!cu_function || gx == 0 || gy == 0 || gz == 0 || bx == 0 || by == 0 || bz == 0) return -EINVAL;
    int rc = gsys_launch_begin((uint64_t)gx * gy * gz, stream);
    if (rc) return rc;
    if (smem_bytes > 48 * 1024 &&
        p_funcsetattr((CUfunction)cu_function, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)smem_bytes) !=
            CUDA_SUCCESS)
        return -EINVAL;
    const CUresult r = p_launch((CUfunction)cu_function, gx, gy, gz, bx, by, bz, (unsigned)smem_bytes,
                                (CUstream)stream, args, nullptr);
    if (r == CUDA_SUCCESS) return 0;
    if (r == CUDA_ERROR_INVALID_VALUE || r == CUDA_ERROR_INVALID_HANDLE) return -EINVAL;
    if (r == CUDA_ERROR_OUT_OF_MEMORY) return -ENOMEM;
    return -EIO;
}

}  // extern "C"
namespace {
struct FlushRec { unsigned long long src, dst; long long ret; const unsigned* consumed; unsigned pos, pad_; };
// gsys_wait's flush of deferred pulls (B15): block b takes record b -- unless a GPU consumer
// (token wait, slot claim) already claimed it -- copies the request's bytes from the host-mapped
// range to its device destination and marks it consumed.
__global__ void flush_kernel(const gsys_dev_ctx* c, const FlushRec* list, unsigned n) {
    __shared__ int s_mine;
    for (unsigned b = blockIdx.x; b < n; b += gridDim.x) {
        const FlushRec f = list[b];
        if (threadIdx.x == 0) s_mine = gsys::claim_record(c, f.pos);
        __syncthreads();
        if (s_mine)
            gsys::pull_copy(reinterpret_cast<const unsigned char*>(f.src), reinterpret_cast<unsigned char*>(f.dst),
                            f.ret, threadIdx.x, blockDim.x);
        __syncthreads();
        if (threadIdx.x == 0 && s_mine)
            asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(f.consumed), "r"(1u) : "memory");
        __syncthreads();
    }
}
}  // namespace

// The flush kernel is launched by service threads while an application kernel may be waiting on
// the service: with lazy module loading its first launch would wait for the running kernels, so
// gsys_init loads it up front.
int preload_flush_kernel() {
    cudaFuncAttributes fa;
    return cudaFuncGetAttributes(&fa, (const void*)flush_kernel) == cudaSuccess ? 0 : -EIO;
}

int Instance::flush_deferred(cudaStream_t st, bool upto_all, uint32_t upto, bool use_kernel, uint64_t only_dst) {
    std::lock_guard<std::mutex> fg(flush_mu);
    std::vector<std::pair<uint32_t, FlushRec>> all;   // (ring position, record)
    const uint32_t h = (uint32_t)head.load(std::memory_order_acquire);
    (void)h;
    for (Worker* w : workers) {
        for (DeferRing* dr : {&w->defer, &w->defer2}) {
            std::lock_guard<std::mutex> g(dr->mu);
            if (!dr->h) continue;
            for (const DeferRing::Region& rg : dr->q) {
                gsys_nbrec& r = nbrec_h[rg.pos & (ring_cap - 1)];
                if (dr->consumed(rg) || !r.src || r.ret <= 0) continue;
                if (!upto_all && (int32_t)(rg.pos - upto) > 0) continue;
                if (only_dst && r.dst != only_dst) continue;
                all.push_back({rg.pos, FlushRec{r.src, r.dst, r.ret, &nbrec_d[rg.pos & (ring_cap - 1)].consumed, rg.pos, 0u}});
            }
        }
    }
    if (all.empty()) return 0;
    // in request order; reads into the same destination go in separate passes, so the last one
    // issued is the one that stays (one caller's back-to-back reads into one buffer)
    std::sort(all.begin(), all.end(), [](const auto& a, const auto& b) { return (int32_t)(a.first - b.first) < 0; });
    if (!use_kernel) {   // copy-engine copies in request order on one stream, then mark consumed
        for (const auto& pr : all)
            cudaMemcpyAsync((void*)pr.second.dst, (const void*)pr.second.src, (size_t)pr.second.ret,
                            cudaMemcpyHostToDevice, st);
        const cudaError_t e = cudaStreamSynchronize(st);
        for (const auto& pr : all)
            __atomic_store_n(&nbrec_h[pr.first & (ring_cap - 1)].consumed, 1u, __ATOMIC_RELEASE);
        st_flushed.fetch_add(all.size(), std::memory_order_relaxed);
        return e == cudaSuccess ? 0 : -EIO;
    }
    // the record list lives in a grow-only pinned buffer: freeing pinned memory synchronises the
    // device, which must not happen here while a kernel may be waiting on this service
    if (flush_cap < all.size()) {
        size_t cap = std::max<size_t>(4096, flush_cap * 2);
        while (cap < all.size()) cap *= 2;
        void* nb = nullptr;
        if (cudaHostAlloc(&nb, cap * sizeof(FlushRec), cudaHostAllocMapped) != cudaSuccess) return -ENOMEM;
        if (flush_buf) flush_old.push_back(flush_buf);   // freed at shutdown
        flush_buf = nb;
        flush_cap = cap;
    }
    FlushRec* lh = (FlushRec*)flush_buf;
    FlushRec* ld = nullptr;
    cudaHostGetDevicePointer((void**)&ld, lh, 0);
    size_t n = 0, start = 0;
    std::unordered_set<unsigned long long> dsts;
    auto launch = [&]() {
        if (n == start) return;
        const unsigned cnt = (unsigned)(n - start);
        flush_kernel<<<std::min<unsigned>(cnt, 4096), 256, 0, st>>>(ctx_d, ld + start, cnt);
        start = n;
        dsts.clear();
    };
    for (const auto& pr : all) {
        if (dsts.count(pr.second.dst)) launch();
        dsts.insert(pr.second.dst);
        lh[n++] = pr.second;
    }
    launch();
    cudaError_t e = cudaStreamSynchronize(st);
    st_flushed.fetch_add(all.size(), std::memory_order_relaxed);
    return e == cudaSuccess ? 0 : -EIO;
}

extern "C" {

int gsys_wait(void* stream) {
    Instance* I = current();
    if (!I) return -ENODEV;
    cudaError_t e = stream ? cudaStreamSynchronize((cudaStream_t)stream) : cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_err(e);
    uint32_t tail = 0;
    gsys_wd_log wd;
    cudaMemcpyAsync(&tail, I->tail_d, 4, cudaMemcpyDeviceToHost, I->ctl);
    cudaMemcpyAsync(&wd, I->wd_d, sizeof wd, cudaMemcpyDeviceToHost, I->ctl);
    cudaStreamSynchronize(I->ctl);
    uint64_t h = I->head.load(std::memory_order_acquire);
    uint64_t issued = h + (uint64_t)(uint32_t)(tail - (uint32_t)h);
    // drain: every published request served and its completion landed (P34.9).  After a watchdog
    // expiry a request may never complete (a lost completion, a call that never returns): then
    // the drain is bounded by the same timeout.
    const uint64_t t0 = now_ns();
    const uint64_t lim = wd.count ? std::max<uint64_t>(I->ctx_h.poll_timeout_ns, 1000000ull) : 0;
    bool drained = true;
    while (I->head.load(std::memory_order_acquire) < issued || I->completed.load(std::memory_order_acquire) < issued) {
        if (lim && now_ns() - t0 > lim) { drained = false; break; }
        std::this_thread::yield();
    }
    for (Worker* w : I->workers) cudaStreamSynchronize(w->stream);
    // deferred pulls nobody waited for on the GPU land now (B15).  Kernels on other streams may
    // still consume records themselves: every GPU copier claims a record in device memory first,
    // so the flush kernel takes only the ones nobody else has
    int ferr = 0;
    if (drained) {
        ferr = I->flush_deferred(I->ctl, true, 0u, true);
        for (Worker* w : I->workers) {
            std::lock_guard<std::mutex> g(w->dmu);
            w->dmap.clear();
        }
    }
    if (ferr) {
        int z = 0;
        I->first_err.compare_exchange_strong(z, ferr);
    }
    if (wd.count) {
        // slots whose waits expired were left claimed (the host might still complete into them);
        // once the service is drained they are returned to free -- every slot after a
        // device-wide wait (no kernel can hold a claim then), else the logged ones
        if (drained) {
            // (the host-visible state word too: a pulled bounce range waits for it, reading B13)
            if (!stream) {
                cudaMemsetAsync(I->claim_d, 0, (size_t)I->nslots * 4, I->ctl);
                cudaMemsetAsync(I->nbpend_d, 0, (size_t)I->nslots * 4, I->ctl);
                for (uint32_t s = 0; s < I->nslots; s++)
                    if (__atomic_load_n(&I->area_h[s].state, __ATOMIC_RELAXED) != GSYS_FREE)
                        __atomic_store_n(&I->area_h[s].state, (uint32_t)GSYS_FREE, __ATOMIC_RELEASE);
            } else {
                for (uint32_t i = 0; i < std::min<uint32_t>(wd.count, GSYS_WD_RECS); i++) {
                    const uint32_t s = wd.rec[i].slot;
                    if (wd.rec[i].phase == GSYS_WD_KERNEL || wd.rec[i].phase == GSYS_WD_CLAIM || s >= I->nslots) continue;
                    cudaMemsetAsync(I->claim_d + s, 0, 4, I->ctl);
                    cudaMemsetAsync(I->nbpend_d + s, 0, 4, I->ctl);
                    __atomic_store_n(&I->area_h[s].state, (uint32_t)GSYS_FREE, __ATOMIC_RELEASE);
                }
            }
        }
        {
            std::lock_guard<std::mutex> g(I->wd_mu);
            I->wd_last = wd;
        }
        cudaMemsetAsync(I->wd_d, 0, sizeof(gsys_wd_log), I->ctl);
        cudaStreamSynchronize(I->ctl);
        I->first_err.store(0);
        return -ETIMEDOUT;
    }
    return I->first_err.exchange(0);
}

int gsys_watchdog_read(uint32_t* count, uint32_t* recs, uint32_t cap) {
    Instance* I = current();
    if (!I) return -ENODEV;
    std::lock_guard<std::mutex> g(I->wd_mu);
    if (count) *count = I->wd_last.count;
    const uint32_t k = std::min<uint32_t>(std::min<uint32_t>(I->wd_last.count, GSYS_WD_RECS), cap);
    for (uint32_t i = 0; recs && i < k; i++) {
        recs[4 * i + 0] = I->wd_last.rec[i].slot;
        recs[4 * i + 1] = I->wd_last.rec[i].seq;
        recs[4 * i + 2] = I->wd_last.rec[i].nr;
        recs[4 * i + 3] = I->wd_last.rec[i].phase;
    }
    return (int)k;
}

int gsys_set_poll_timeout(uint32_t ms) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (cudaDeviceSynchronize() != cudaSuccess) return -EIO;   // running kernels read the context
    I->ctx_h.poll_timeout_ns = (unsigned long long)ms * 1000000ull;
    if (cudaMemcpy(I->ctx_d, &I->ctx_h, sizeof I->ctx_h, cudaMemcpyHostToDevice) != cudaSuccess) return -EIO;
    return 0;
}

// ---------------------------------------------------------------- clock relation (trace timestamps)
}  // extern "C"
namespace {
// One thread: measure the %globaltimer tick, then `samples` ping-pongs with the host through
// host-mapped words; t[2i], t[2i+1] = GPU time before the ping and after the pong.
__global__ void clock_sync_kernel(unsigned* ping, const unsigned* pong, unsigned long long* t, unsigned samples,
                                  unsigned long long* tick) {
    unsigned long long prev = gsys::globaltimer(), best = ~0ull;
    for (int i = 0; i < 20000 && best > 1; i++) {
        const unsigned long long x = gsys::globaltimer();
        if (x != prev) { if (x - prev < best) best = x - prev; prev = x; }
    }
    *tick = best;
    for (unsigned i = 1; i <= samples; i++) {
        const unsigned long long g0 = gsys::globaltimer();
        asm volatile("st.release.sys.global.u32 [%0], %1;" :: "l"(ping), "r"(i) : "memory");
        const unsigned long long tlim = g0 + 1000000000ull;
        unsigned v;
        do {
            asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(pong) : "memory");
        } while (v != i && gsys::globaltimer() < tlim);
        t[2 * i - 2] = g0;
        t[2 * i - 1] = v == i ? gsys::globaltimer() : 0ull;
        if (v != i) return;
    }
}
}  // namespace
extern "C" {

int gsys_clock_sync(uint32_t samples, int64_t* offset_ns, uint64_t* uncertainty_ns) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (samples == 0 || samples > 4096 || !offset_ns || !uncertainty_ns) return -EINVAL;
    const size_t bytes = 256 + 16ull * samples;
    uint8_t* buf = nullptr;
    if (cudaHostAlloc((void**)&buf, bytes, cudaHostAllocMapped) != cudaSuccess) return -ENOMEM;
    memset(buf, 0, bytes);
    uint8_t* dbuf = nullptr;
    cudaHostGetDevicePointer((void**)&dbuf, buf, 0);
    volatile unsigned* ping = (volatile unsigned*)buf;
    volatile unsigned* pong = (volatile unsigned*)(buf + 64);
    unsigned long long* tick = (unsigned long long*)(buf + 128);
    unsigned long long* t = (unsigned long long*)(buf + 256);
    std::vector<uint64_t> h(samples, 0);
    clock_sync_kernel<<<1, 1, 0, I->ctl>>>((unsigned*)dbuf, (const unsigned*)(dbuf + 64),
                                           (unsigned long long*)(dbuf + 256), samples,
                                           (unsigned long long*)(dbuf + 128));
    int rc = cuda_err(cudaGetLastError());
    for (uint32_t i = 1; rc == 0 && i <= samples; i++) {
        const uint64_t tl = now_ns() + 1000000000ull;
        while (__atomic_load_n(ping, __ATOMIC_ACQUIRE) != i) {
            if (now_ns() > tl) { rc = -ETIMEDOUT; break; }
        }
        if (rc) break;
        h[i - 1] = now_ns();
        __atomic_store_n(pong, i, __ATOMIC_RELEASE);
    }
    if (cudaStreamSynchronize(I->ctl) != cudaSuccess && rc == 0) rc = -EIO;
    if (rc == 0) {
        uint64_t best = ~0ull;
        for (uint32_t i = 0; i < samples; i++) {
            const uint64_t g0 = t[2 * i], g1 = t[2 * i + 1];
            if (!g1 || g1 < g0) continue;
            if (g1 - g0 < best) {
                best = g1 - g0;
                *offset_ns = (int64_t)(h[i] - (g0 + (g1 - g0) / 2));
            }
        }
        if (best == ~0ull) rc = -EIO;
        else *uncertainty_ns = best / 2 + *tick;
    }
    cudaFreeHost(buf);
    return rc;
}

int gsys_set_completion(uint32_t mode) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (mode > GSYS_COMPLETION_PULL) return -EINVAL;
    if (cudaDeviceSynchronize() != cudaSuccess) return -EIO;   // running kernels read the context
    // (requests carry their completion path in their flags: the service needs no drain here)
    I->ctx_h.memop_completion = mode == GSYS_COMPLETION_MEMOP ? 1u : 0u;
    I->ctx_h.pull_bounce = mode == GSYS_COMPLETION_PULL ? 1u : 0u;
    I->memop_completion = I->ctx_h.memop_completion != 0;
    if (cudaMemcpy(I->ctx_d, &I->ctx_h, sizeof I->ctx_h, cudaMemcpyHostToDevice) != cudaSuccess) return -EIO;
    return 0;
}

int gsys_set_fault_drop(int64_t offset) {
    Instance* I = current();
    if (!I) return -ENODEV;
    I->drop_off.store(offset < 0 ? -1 : offset);
    return 0;
}

int gsys_shutdown(void) {
    std::lock_guard<std::mutex> g(g_mu);
    int d = 0;
    if (cudaGetDevice(&d) != cudaSuccess || d < 0 || d >= 64) return 0;
    Instance* I = g_inst[d];
    if (!I) return 0;
    int r = gsys_wait(nullptr);
    I->stop.store(true);
    {
        std::lock_guard<std::mutex> lk(I->sleep_mu);
        I->sleep_cv.notify_all();
    }
    for (Worker* w : I->workers) {
        if (w->th.joinable()) w->th.join();
        cudaStreamSynchronize(w->stream);
        w->ring->drain();
        delete w->ring;
        for (auto e : w->evpool) cudaEventDestroy(e);
        cudaStreamDestroy(w->stream);
        cudaFreeHost(w->bounce);
        if (w->defer.h) cudaFreeHost(w->defer.h);
        if (w->defer2.h) cudaFreeHost(w->defer2.h);
        delete w;
    }
    cudaFreeHost(I->area_h);
    cudaFreeHost(I->inline_h);
    if (I->pull_h) cudaFreeHost(I->pull_h);
    cudaFreeHost(I->ring_h);
    cudaFreeHost(I->hdone_h);
    cudaFreeHost(I->nbrec_h);
    if (I->flush_buf) cudaFreeHost(I->flush_buf);
    for (void* p : I->flush_old) cudaFreeHost(p);
    cudaFree(I->claim_d);
    cudaFree(I->seqs_d);
    cudaFree(I->mirror_d);
    cudaFree(I->tail_d);
    cudaFree(I->lat_hint_d);
    cudaFree(I->nbpend_d);
    cudaFree(I->nbpos_d);
    cudaFree(I->nbclaim_d);
    cudaFree(I->krounds_d);
    cudaFree(I->kblock_d);
    cudaFree(I->ctx_d);
    cudaFree(I->wd_d);
    if (I->gtrace_d) cudaFree(I->gtrace_d);
    if (I->gtrace_n_d) cudaFree(I->gtrace_n_d);
    for (void* p : I->graveyard) cudaFree(p);
    cudaStreamDestroy(I->ctl);
    g_inst[d] = nullptr;
    delete I;
    return r;
}

const void* gsys_device_ctx(void) {
    Instance* I = current();
    return I ? (const void*)I->ctx_d : nullptr;
}

int gsys_stats(gsys_stats_t* out) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (!out) return -EINVAL;
    memset(out, 0, sizeof *out);
    out->requests = I->head.load();
    out->completed = I->completed.load();
    out->bundles = I->st_bundles.load();
    out->max_bundle = I->st_max_bundle.load();
    out->host_preads = I->st_host_preads.load();
    out->merged = I->st_merged.load();
    out->bytes_read = I->st_bytes_read.load();
    out->bytes_h2d = I->st_bytes_h2d.load();
    out->errors = I->st_errors.load();
    for (int k = 0; k < 8; k++) out->per_nr[k] = I->st_nr[k].load();
    out->ns_busy = I->st_ns_busy.load();
    out->ns_syscall = I->st_ns_syscall.load();
    out->ns_cuda = I->st_ns_cuda.load();
    out->ns_bounce_wait = I->st_ns_wait.load();
    out->threads = I->nthreads;
    out->slots = I->nslots;
    out->coalesce_max = I->coalesce_max.load();
    out->coalesce_window_us = I->window_us.load();
    out->split = I->st_split.load();
    out->deferred = I->st_deferred.load();
    out->flushed = I->st_flushed.load();
    return 0;
}

int gsys_stats_reset(void) {
    Instance* I = current();
    if (!I) return -ENODEV;
    I->st_bundles.store(0);
    I->st_max_bundle.store(0);
    I->st_ns_busy.store(0);
    I->st_ns_syscall.store(0);
    I->st_ns_cuda.store(0);
    I->st_ns_wait.store(0);
    I->st_host_preads.store(0);
    I->st_merged.store(0);
    I->st_bytes_read.store(0);
    I->st_bytes_h2d.store(0);
    I->st_errors.store(0);
    I->st_split.store(0);
    I->st_deferred.store(0);
    I->st_flushed.store(0);
    for (auto& a : I->st_nr) a.store(0);
    return 0;
}

int gsys_abi_info(uint32_t* slot_bytes, uint32_t* inline_bytes, uint32_t* nstates) {
    if (slot_bytes) *slot_bytes = (uint32_t)sizeof(gsys_slot);
    if (inline_bytes) *inline_bytes = GSYS_INLINE_BYTES;
    if (nstates) *nstates = 5;
    return 0;
}

// Merge planner (reading A8): stable sort by (fd, off), then grow a group while the next request
// is on the same fd, starts at or before the current union end (adjacent or overlapping), and the
// union stays within max_union bytes.
int gsys_plan_merge(uint32_t n, const int32_t* fd, const int64_t* off, const uint64_t* len, uint64_t max_union,
                    uint32_t* order, uint32_t* group, uint64_t* offset_in_group, int64_t* group_off,
                    uint64_t* group_len) {
    if (n == 0) return 0;
    if (!fd || !off || !len || !order || !group || !offset_in_group || !group_off || !group_len) return -EINVAL;
    for (uint32_t i = 0; i < n; i++) order[i] = i;
    std::stable_sort(order, order + n, [&](uint32_t a, uint32_t b) {
        if (fd[a] != fd[b]) return fd[a] < fd[b];
        return off[a] < off[b];
    });
    int g = -1;
    int64_t u0 = 0, u1 = 0;
    int32_t gfd = 0;
    for (uint32_t t = 0; t < n; t++) {
        uint32_t i = order[t];
        int64_t lo = off[i], hi = off[i] + (int64_t)len[i];
        bool join = g >= 0 && fd[i] == gfd && lo >= 0 && lo <= u1 &&
                    (uint64_t)(std::max(u1, hi) - u0) <= max_union && len[i] > 0;
        if (!join) {
            g++;
            gfd = fd[i];
            u0 = lo;
            u1 = hi;
        } else {
            u1 = std::max(u1, hi);
        }
        group[i] = (uint32_t)g;
        offset_in_group[i] = (uint64_t)(lo - u0);
        group_off[g] = u0;
        group_len[g] = (uint64_t)(u1 - u0);
    }
    return g + 1;
}

// ---------------------------------------------------------------- signal sink (config 5b)
// A process-directed signal may land on any thread of the process (PyTorch owns several), so the
// consumer side is an async-signal-safe SA_SIGINFO handler that appends si_value to a ring; the
// application drains it with gsys_sigsink_read().
namespace {
std::atomic<uint64_t> g_sig_head{0}, g_sig_tail{0};
int32_t* g_sig_ring = nullptr;
uint64_t* g_sig_ts = nullptr;
uint32_t g_sig_cap = 0;
std::atomic<uint64_t> g_sig_dropped{0};

void sigsink_handler(int, siginfo_t* si, void*) {
    // reserve an entry only while the ring has room (a dropped signal must not leave a hole the
    // reader would stop at forever)
    const uint32_t cap = __atomic_load_n(&g_sig_cap, __ATOMIC_ACQUIRE);   // 0 while re-installing
    int32_t* const ring = g_sig_ring;
    uint64_t* const tsb = g_sig_ts;
    uint64_t i = g_sig_tail.load(std::memory_order_relaxed);
    do {
        if (cap == 0 || i - g_sig_head.load(std::memory_order_acquire) >= cap) {
            g_sig_dropped.fetch_add(1, std::memory_order_relaxed);
            return;
        }
    } while (!g_sig_tail.compare_exchange_weak(i, i + 1, std::memory_order_acq_rel));
    struct timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    tsb[i % cap] = (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
    __atomic_store_n(&ring[i % cap], si->si_value.sival_int, __ATOMIC_RELEASE);
}
}  // namespace

int gsys_sigsink_install(int32_t sig, uint32_t capacity) {
    if (sig < SIGRTMIN || sig > SIGRTMAX || capacity == 0) return -EINVAL;
    if (!g_sig_ring || capacity > g_sig_cap) {
        // (re)allocate with `sig` blocked in this thread; the previous ring must be drained -- a
        // larger request replaces it only when no signal is pending in it
        if (g_sig_ring && g_sig_tail.load() != g_sig_head.load()) return -EBUSY;
        sigset_t ss, old;
        sigemptyset(&ss);
        sigaddset(&ss, sig);
        pthread_sigmask(SIG_BLOCK, &ss, &old);
        int32_t* ring = (int32_t*)calloc(capacity, sizeof(int32_t));
        uint64_t* tsb = (uint64_t*)calloc(capacity, sizeof(uint64_t));
        if (!ring || !tsb) {
            free(ring);
            free(tsb);
            pthread_sigmask(SIG_SETMASK, &old, nullptr);
            return -ENOMEM;
        }
        for (uint32_t i = 0; i < capacity; i++) ring[i] = INT32_MIN;
        // handlers on other threads drop while the cap is 0; the previous ring is not freed (a
        // handler on another thread may still hold its pointer)
        __atomic_store_n(&g_sig_cap, 0u, __ATOMIC_RELEASE);
        g_sig_ring = ring;
        g_sig_ts = tsb;
        g_sig_head.store(0);
        g_sig_tail.store(0);
        __atomic_store_n(&g_sig_cap, capacity, __ATOMIC_RELEASE);
        pthread_sigmask(SIG_SETMASK, &old, nullptr);
    }
    struct sigaction sa;
    memset(&sa, 0, sizeof sa);
    sa.sa_sigaction = sigsink_handler;
    sa.sa_flags = SA_SIGINFO | SA_RESTART;
    sigemptyset(&sa.sa_mask);
    return sigaction(sig, &sa, nullptr) == 0 ? 0 : -errno;
}

int gsys_sigsink_read(int32_t* values, uint64_t* t_ns, uint32_t cap) {
    if (!g_sig_ring) return -ENODEV;
    uint32_t n = 0;
    uint64_t h = g_sig_head.load(std::memory_order_relaxed);
    const uint64_t t = g_sig_tail.load(std::memory_order_acquire);
    const uint32_t rc = __atomic_load_n(&g_sig_cap, __ATOMIC_ACQUIRE);
    if (rc == 0) return 0;
    while (h < t && n < cap) {
        int32_t v = __atomic_load_n(&g_sig_ring[h % rc], __ATOMIC_ACQUIRE);
        if (v == INT32_MIN) break;   // slot claimed by a handler that has not stored yet
        values[n] = v;
        if (t_ns) t_ns[n] = g_sig_ts[h % rc];
        g_sig_ring[h % rc] = INT32_MIN;
        n++;
        h++;
    }
    g_sig_head.store(h, std::memory_order_release);
    return (int)n;
}

// Self-test of the bounce ring allocator with a fake completion model: random allocation sizes
// and commit points; after every allocation no other in-flight region may overlap the new one,
// and every waited token must have been issued.  Returns 0 or -EPROTO.
namespace {
struct FakeOps {
    uint64_t issued = 0, waited_max = 0, waits = 0;
    bool bad = false;
    uint64_t make_token() { return ++issued; }
    void wait(uint64_t t) {
        if (t == 0 || t > issued) bad = true;
        waits++;
        if (t > waited_max) waited_max = t;
    }
    void recycle(uint64_t) {}
};
}  // namespace

int gsys_selftest_bounce(uint64_t seed, uint32_t iters, uint64_t cap) {
    if (cap < 4096) return -EINVAL;
    FakeOps ops;
    BounceRing<uint64_t, FakeOps> ring(cap, &ops);
    uint64_t x = seed | 1;
    for (uint32_t i = 0; i < iters; i++) {
        x ^= x << 13; x ^= x >> 7; x ^= x << 17;
        size_t n = 1 + (size_t)(x % (cap / ((x >> 20) % 4 == 0 ? 1 : 8)));
        size_t lo = ring.alloc(n);
        if (n > cap) { if (lo != ring.NONE) return -EPROTO; continue; }
        if (lo == ring.NONE) return -EPROTO;
        size_t hi = lo + ((n + 255) & ~(size_t)255);
        if (hi > cap || !ring.disjoint_from_inflight(lo, hi)) return -EPROTO;
        if ((x >> 33) % 3 == 0) ring.commit();
    }
    ring.drain();
    return ops.bad ? -EPROTO : 0;
}

int64_t gsys_split_result(int64_t r, uint64_t offset_in_group, uint64_t len) {
    if (r < 0) return r;
    int64_t v = r - (int64_t)offset_in_group;
    if (v < 0) v = 0;
    if ((uint64_t)v > len) v = (int64_t)len;
    return v;
}

}  // extern "C"
