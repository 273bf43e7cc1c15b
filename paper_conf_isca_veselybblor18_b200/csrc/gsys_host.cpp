// gsys_host.cpp -- host half of libgsys: syscall area, doorbell drain, coalescing, execution.
//
// Replaces GENESYS's kernel-side processing (sec. VI "CPU-side system call
// processing", P24.16-35) with a user-space service, because the box's kernel cannot be changed
// (BASELINE.json north_star):
//   * the paper's interrupt handler, which "creates a new kernel task and adds it to Linux's
//     work-queue" after "waiting for a predetermined amount of time" to coalesce (P24.17-18,
//     P24.29-30), becomes ONE dispatcher thread per GPU that polls the doorbell ring the GPU
//     writes (the s_sendmsg analogue, P24.14) and cuts the entries into bundles of at most
//     coalesce_max requests or coalesce_window microseconds (P22.9-13);
//   * the "OS worker thread" that "atomically switches any ready system call requests to the
//     processing state" and "carries out the system call work" (P24.19-21) becomes a pool of
//     worker threads that execute a bundle in (fd, offset) order (reading A8), merge preads of
//     adjacent/overlapping ranges into one read of the union (north_star extension), DMA payloads
//     into device buffers and publish results (P24.32-35);
//   * results are returned with CUDA stream memory operations ordered after the payload DMA:
//     blocking -> completion word {seq, ret} (state "finished"), non-blocking -> claim word
//     cleared (state "free"), P24.33-34;
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
#include <mutex>
#include <numeric>
#include <thread>
#include <vector>

#include "gsys.h"
#include "gsys_device.cuh"
#include "gsys_internal.h"

namespace {

typedef CUresult (*PFN_batch_t)(CUstream, unsigned int, CUstreamBatchMemOpParams*, unsigned int);
typedef CUresult (*PFN_ptrattrs_t)(unsigned int, CUpointer_attribute*, void**, CUdeviceptr);
typedef CUresult (*PFN_devattr_t)(int*, CUdevice_attribute, CUdevice);

PFN_batch_t p_batch = nullptr;
PFN_ptrattrs_t p_ptrattrs = nullptr;
PFN_devattr_t p_devattr = nullptr;

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

// ------------------------------------------------------------------ bounded MPMC queue (Vyukov)
class MPMC {
   public:
    explicit MPMC(size_t cap_pow2) : mask_(cap_pow2 - 1), cells_(cap_pow2) {
        for (size_t i = 0; i < cap_pow2; i++) cells_[i].seq.store(i, std::memory_order_relaxed);
        enq_.store(0); deq_.store(0);
    }
    bool push(uint64_t v) {
        size_t pos = enq_.load(std::memory_order_relaxed);
        for (;;) {
            Cell& c = cells_[pos & mask_];
            size_t seq = c.seq.load(std::memory_order_acquire);
            intptr_t d = (intptr_t)seq - (intptr_t)pos;
            if (d == 0) {
                if (enq_.compare_exchange_weak(pos, pos + 1, std::memory_order_relaxed)) {
                    c.val = v;
                    c.seq.store(pos + 1, std::memory_order_release);
                    return true;
                }
            } else if (d < 0) {
                return false;
            } else {
                pos = enq_.load(std::memory_order_relaxed);
            }
        }
    }
    bool pop(uint64_t* v) {
        size_t pos = deq_.load(std::memory_order_relaxed);
        for (;;) {
            Cell& c = cells_[pos & mask_];
            size_t seq = c.seq.load(std::memory_order_acquire);
            intptr_t d = (intptr_t)seq - (intptr_t)(pos + 1);
            if (d == 0) {
                if (deq_.compare_exchange_weak(pos, pos + 1, std::memory_order_relaxed)) {
                    *v = c.val;
                    c.seq.store(pos + mask_ + 1, std::memory_order_release);
                    return true;
                }
            } else if (d < 0) {
                return false;
            } else {
                pos = deq_.load(std::memory_order_relaxed);
            }
        }
    }

   private:
    struct alignas(64) Cell {
        std::atomic<size_t> seq;
        uint64_t val;
    };
    size_t mask_;
    std::vector<Cell> cells_;
    alignas(64) std::atomic<size_t> enq_;
    alignas(64) std::atomic<size_t> deq_;
};

enum PtrKind { PK_INVALID = 0, PK_DEVICE = 1, PK_HOST = 2 };

struct Instance;

struct Req {
    uint32_t slot, seq, nr, flags;
    uint64_t a[6];
    int64_t ret;
    bool ok;
};

// ------------------------------------------------------------------ worker
struct Worker {
    Instance* inst = nullptr;
    int id = 0;
    std::thread th;
    cudaStream_t stream = nullptr;
    uint8_t* bounce = nullptr;       // pinned
    size_t bcap = 0, bhead = 0;
    struct Region { size_t lo, hi; cudaEvent_t ev; bool last; };
    std::deque<Region> inflight;
    std::vector<size_t> pending;      // indices into `inflight` awaiting an event (uncommitted)
    std::vector<cudaEvent_t> evpool;
    std::vector<Req> reqs;
    std::vector<CUstreamBatchMemOpParams> ops;
    struct Cache { uintptr_t lo, hi; PtrKind kind; intptr_t host_delta; uint64_t gen; };
    std::vector<Cache> cache;
    // merge scratch
    std::vector<int32_t> mfd; std::vector<int64_t> moff; std::vector<uint64_t> mlen;
    std::vector<uint32_t> morder, mgroup; std::vector<uint64_t> mgoff_in; std::vector<int64_t> mg_off;
    std::vector<uint64_t> mg_len; std::vector<uint32_t> midx;

    cudaEvent_t get_event() {
        if (!evpool.empty()) { cudaEvent_t e = evpool.back(); evpool.pop_back(); return e; }
        cudaEvent_t e;
        cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
        return e;
    }
    // allocate n bytes of pinned bounce, waiting for in-flight DMA that still reads the range
    uint8_t* alloc(size_t n) {
        n = (n + 255) & ~(size_t)255;
        if (n > bcap) return nullptr;
        if (bhead + n > bcap) bhead = 0;
        size_t lo = bhead, hi = bhead + n;
        while (!inflight.empty()) {
            Region& f = inflight.front();
            bool overlap = f.lo < hi && lo < f.hi;
            if (!overlap) break;
            if (f.ev) {
                cudaEventSynchronize(f.ev);
                if (f.last) evpool.push_back(f.ev);
            } else {
                // uncommitted region of the current bundle: commit first, then wait
                commit();
                continue;
            }
            inflight.pop_front();
            for (auto& p : pending) p--;   // indices shift
        }
        inflight.push_back(Region{lo, hi, nullptr, false});
        pending.push_back(inflight.size() - 1);
        bhead = hi;
        return bounce + lo;
    }
    // record one event after the copies issued so far and attach it to uncommitted regions
    void commit() {
        if (pending.empty()) return;
        cudaEvent_t e = get_event();
        cudaEventRecord(e, stream);
        for (size_t i = 0; i < pending.size(); i++) {
            inflight[pending[i]].ev = e;
            inflight[pending[i]].last = (i + 1 == pending.size());
        }
        pending.clear();
    }
    PtrKind resolve(uintptr_t p, size_t n, uint8_t** host);
    void run();
    void process(uint64_t h0, uint32_t n);
    int64_t do_pread(Req& r);
    int64_t do_pwrite(Req& r);
    int64_t do_getrusage(Req& r);
    int64_t do_generic(Req& r);
    int read_small(uintptr_t p, void* out, size_t n);
    int write_small(uintptr_t p, const void* in, size_t n);
    void h2d(void* dst, const void* src, size_t n) {
        cudaMemcpyAsync(dst, src, n, cudaMemcpyHostToDevice, stream);
    }
};

// ------------------------------------------------------------------ instance
struct Instance {
    int dev = -1;
    uint32_t nslots = 0;
    gsys_slot* area_h = nullptr;        // pinned, mapped
    gsys_slot* area_d = nullptr;
    uint8_t* inline_h = nullptr;
    uint8_t* inline_d = nullptr;
    uint64_t* ring_h = nullptr;
    uint64_t* ring_d = nullptr;
    uint32_t ring_cap = 0;
    uint32_t* claim_d = nullptr;
    uint32_t* seqs_d = nullptr;
    unsigned long long* mirror_d = nullptr;
    uint32_t* tail_d = nullptr;
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

    // service
    std::thread dispatcher;
    std::vector<Worker*> workers;
    MPMC* queue = nullptr;
    std::atomic<bool> stop{false};
    std::atomic<uint64_t> head{0};         // doorbell entries consumed (dispatcher)
    std::atomic<uint64_t> completed{0};    // requests whose completion was issued
    std::atomic<int> first_err{0};
    std::atomic<uint32_t> coalesce_max{8};
    std::atomic<uint32_t> window_us{0};
    std::atomic<int> merge{1};
    std::atomic<uint64_t> gen{1};          // pointer-cache generation
    std::atomic<uint64_t> kick{0};
    std::mutex sleep_mu;
    std::condition_variable sleep_cv;
    std::atomic<int> sleepers{0};
    uint32_t nthreads = 0;

    // stats
    std::atomic<uint64_t> st_bundles{0}, st_max_bundle{0}, st_host_preads{0}, st_merged{0},
        st_bytes_read{0}, st_bytes_h2d{0}, st_errors{0};
    std::atomic<uint64_t> st_nr[8];

    // host trace
    std::atomic<int> tracing{0};
    std::mutex trace_mu;
    std::vector<gsys_trace_rec> htrace;

    Instance() { for (auto& a : st_nr) a.store(0); }

    void host_trace(uint32_t s, uint32_t seq, uint8_t from, uint8_t to, bool blocking) {
        if (!tracing.load(std::memory_order_relaxed)) return;
        std::lock_guard<std::mutex> g(trace_mu);
        if (htrace.size() < trace_cap) {
            gsys_trace_rec r;
            r.slot = s; r.seq = seq; r.from = from; r.to = to; r.actor = 1; r.blocking = blocking ? 1 : 0; r.pad = 0;
            htrace.push_back(r);
        }
    }
    void dispatch_loop();
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

// ------------------------------------------------------------------ dispatcher (interrupt-handler analogue)
void Instance::dispatch_loop() {
    cudaSetDevice(dev);
    const uint32_t mask = ring_cap - 1;
    uint64_t h = head.load();
    uint64_t idle_since = now_ns();
    uint64_t last_kick = kick.load();
    auto ready = [&](uint64_t pos) -> bool {
        uint64_t v = __atomic_load_n(&ring_h[pos & mask], __ATOMIC_ACQUIRE);
        return (uint32_t)(v >> 32) == (uint32_t)(pos + 1);
    };
    while (!stop.load(std::memory_order_relaxed)) {
        if (!ready(h)) {
            uint64_t k = kick.load(std::memory_order_relaxed);
            if (k != last_kick) { last_kick = k; idle_since = now_ns(); }
            if (now_ns() - idle_since > 5000000ull) {
                struct timespec ts = {0, 20000};
                nanosleep(&ts, nullptr);
            } else {
                _mm_pause();
            }
            continue;
        }
        // first entry of a bundle: the coalescing window starts now (reading A19)
        uint64_t h0 = h;
        uint32_t cmax = coalesce_max.load(std::memory_order_relaxed);
        uint64_t win = (uint64_t)window_us.load(std::memory_order_relaxed) * 1000ull;
        uint64_t t0 = win ? now_ns() : 0;
        h++;
        while (h - h0 < cmax) {
            if (ready(h)) { h++; continue; }
            if (!win || now_ns() - t0 >= win) break;
            _mm_pause();
        }
        uint32_t n = (uint32_t)(h - h0);
        while (!queue->push((h0 << 16) | (uint64_t)(n - 1))) _mm_pause();
        head.store(h, std::memory_order_release);
        st_bundles.fetch_add(1, std::memory_order_relaxed);
        uint64_t mb = st_max_bundle.load(std::memory_order_relaxed);
        while (n > mb && !st_max_bundle.compare_exchange_weak(mb, n)) {}
        if (sleepers.load(std::memory_order_relaxed) > 0) {
            std::lock_guard<std::mutex> g(sleep_mu);
            sleep_cv.notify_one();
        }
        idle_since = now_ns();
    }
}

// ------------------------------------------------------------------ worker (OS worker-thread analogue)
void Worker::run() {
    cudaSetDevice(inst->dev);
    uint64_t idle_since = now_ns();
    uint64_t item;
    while (!inst->stop.load(std::memory_order_relaxed)) {
        if (inst->queue->pop(&item)) {
            uint64_t h0 = item >> 16;
            uint32_t n = (uint32_t)(item & 0xffff) + 1;
            process(h0, n);
            idle_since = now_ns();
            continue;
        }
        if (now_ns() - idle_since > 2000000ull) {
            std::unique_lock<std::mutex> lk(inst->sleep_mu);
            inst->sleepers.fetch_add(1);
            inst->sleep_cv.wait_for(lk, std::chrono::microseconds(500));
            inst->sleepers.fetch_sub(1);
        } else {
            _mm_pause();
        }
    }
}

PtrKind Worker::resolve(uintptr_t p, size_t n, uint8_t** host) {
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
    PtrKind k = resolve(buf, n, &hp);
    if (k == PK_INVALID) return -EFAULT;
    inst->st_host_preads.fetch_add(1, std::memory_order_relaxed);
    if (k == PK_HOST) {
        ssize_t z = pread(fd, hp, n, off);
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
        ssize_t z = pread(fd, b, piece, off + (int64_t)total);
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
        if (getrusage(who, &ru) != 0) return -(int64_t)errno;
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
            if (r.a[2] && read_small((uintptr_t)r.a[2], &si, sizeof si) != 0) return -EFAULT;
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
        case GSYS_NR_RECVFROM: {
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
            uint8_t* dst = hp;
            if (k == PK_DEVICE) {
                dst = alloc(n ? n : 1);
                if (!dst) return -ENOMEM;
            }
            ssize_t z = recvfrom((int)r.a[0], dst, n, (int)r.a[3], r.a[4] ? (struct sockaddr*)sa : nullptr,
                                 r.a[5] ? &salen : nullptr);
            if (z < 0) return -(int64_t)errno;
            if (k == PK_DEVICE && z > 0) h2d((void*)r.a[1], dst, (size_t)z);
            if (r.a[4] && write_small((uintptr_t)r.a[4], sa, salen) != 0) return -EFAULT;
            if (r.a[5]) {
                uint32_t l = salen;
                if (write_small((uintptr_t)r.a[5], &l, 4) != 0) return -EFAULT;
            }
            return z;
        }
        default:
            return -ENOSYS;
    }
}

void Worker::process(uint64_t h0, uint32_t n) {
    Instance* I = inst;
    const uint32_t mask = I->ring_cap - 1;
    reqs.resize(n);
    for (uint32_t i = 0; i < n; i++) {
        uint64_t e = __atomic_load_n(&I->ring_h[(h0 + i) & mask], __ATOMIC_ACQUIRE);
        Req& r = reqs[i];
        r.slot = (uint32_t)e;
        volatile gsys_slot* sl = (volatile gsys_slot*)(I->area_h + r.slot);
        r.nr = sl->nr;
        r.flags = sl->flags;
        r.seq = sl->seq;
        for (int k = 0; k < 6; k++) r.a[k] = sl->args[k];
        r.ret = 0;
        // "atomically switches any ready system call requests to the processing state" (P24.20)
        uint32_t expect = GSYS_READY;
        r.ok = __atomic_compare_exchange_n((uint32_t*)&I->area_h[r.slot].state, &expect, (uint32_t)GSYS_PROCESSING,
                                           false, __ATOMIC_ACQ_REL, __ATOMIC_ACQUIRE);
        if (!r.ok) r.ret = -EPROTO;
        I->host_trace(r.slot, r.seq, GSYS_READY, GSYS_PROCESSING, !(r.flags & GSYS_NONBLOCKING));
        I->st_nr[nr_index(r.nr)].fetch_add(1, std::memory_order_relaxed);
    }

    // ---- execute: preads first through the merge planner (reading A8), then the rest in order
    midx.clear();
    for (uint32_t i = 0; i < n; i++)
        if (reqs[i].ok && reqs[i].nr == GSYS_NR_PREAD64) midx.push_back(i);
    std::vector<bool> done(n, false);
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
        std::vector<std::vector<uint32_t>> members(ng > 0 ? ng : 0);
        for (uint32_t t = 0; t < m; t++) members[mgroup[morder[t]]].push_back(morder[t]);
        for (int g = 0; g < ng; g++) {
            auto& mem = members[g];
            if (mem.size() < 2) continue;
            int fd = mfd[mem[0]];
            struct stat st;
            if (fstat(fd, &st) != 0 || !S_ISREG(st.st_mode)) continue;
            bool okd = true;
            for (uint32_t j : mem) {
                Req& r = reqs[midx[j]];
                if (r.a[2] == 0 || resolve((uintptr_t)r.a[1], r.a[2], nullptr) == PK_INVALID) { okd = false; break; }
            }
            if (!okd) continue;
            uint8_t* b = alloc(mg_len[g]);
            if (!b) continue;
            ssize_t z = pread(fd, b, mg_len[g], mg_off[g]);
            I->st_host_preads.fetch_add(1, std::memory_order_relaxed);
            int64_t zr = z < 0 ? -(int64_t)errno : (int64_t)z;
            if (zr > 0) I->st_bytes_read.fetch_add((uint64_t)zr, std::memory_order_relaxed);
            for (uint32_t j : mem) {
                Req& r = reqs[midx[j]];
                int64_t ri = gsys_split_result(zr, mgoff_in[j], r.a[2]);
                r.ret = ri;
                done[midx[j]] = true;
                if (ri > 0) {
                    uint8_t* hp = nullptr;
                    PtrKind k = resolve((uintptr_t)r.a[1], r.a[2], &hp);
                    if (k == PK_HOST) {
                        memcpy(hp, b + mgoff_in[j], (size_t)ri);
                    } else {
                        h2d((void*)r.a[1], b + mgoff_in[j], (size_t)ri);
                        I->st_bytes_h2d.fetch_add((uint64_t)ri, std::memory_order_relaxed);
                    }
                }
            }
            I->st_merged.fetch_add(mem.size(), std::memory_order_relaxed);
        }
        // remaining preads in (fd, off) order
        for (uint32_t t = 0; t < m; t++) {
            uint32_t i = midx[morder[t]];
            if (done[i]) continue;
            reqs[i].ret = do_pread(reqs[i]);
            done[i] = true;
        }
    }
    for (uint32_t i = 0; i < n; i++) {
        Req& r = reqs[i];
        if (!r.ok || done[i]) continue;
        switch (r.nr) {
            case GSYS_NR_PREAD64: r.ret = do_pread(r); break;
            case GSYS_NR_PWRITE64: r.ret = do_pwrite(r); break;
            case GSYS_NR_GETRUSAGE: r.ret = do_getrusage(r); break;
            default: r.ret = do_generic(r); break;
        }
    }

    // ---- completion (P24.32-35): result into args[0]; blocking -> finished + completion word,
    // non-blocking -> free + claim word cleared.  Stream memops are ordered after the DMA above.
    ops.clear();
    for (uint32_t i = 0; i < n; i++) {
        Req& r = reqs[i];
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
            if (r.ok) {
                __atomic_store_n(&sl->state, (uint32_t)GSYS_FINISHED, __ATOMIC_RELEASE);
                I->host_trace(r.slot, r.seq, GSYS_PROCESSING, GSYS_FINISHED, true);
            }
            uint64_t word = ((uint64_t)r.seq << 32) | (uint32_t)(int32_t)r.ret;
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
            if (r.ok) {
                __atomic_store_n(&sl->state, (uint32_t)GSYS_FREE, __ATOMIC_RELEASE);
                I->host_trace(r.slot, r.seq, GSYS_PROCESSING, GSYS_FREE, false);
            }
            op.writeValue.operation = CU_STREAM_MEM_OP_WRITE_VALUE_32;
            op.writeValue.address = (CUdeviceptr)(I->claim_d + r.slot);
            op.writeValue.value = 0;
            op.writeValue.flags = CU_STREAM_WRITE_VALUE_DEFAULT;
            ops.push_back(op);
        }
    }
    for (size_t i = 0; i < ops.size(); i += 128) {
        unsigned cnt = (unsigned)std::min<size_t>(128, ops.size() - i);
        CUresult cr = p_batch((CUstream)stream, cnt, ops.data() + i, 0);
        if (cr != CUDA_SUCCESS) {
            fprintf(stderr, "gsys: cuStreamBatchMemOp failed (%d)\n", (int)cr);
            int z = 0;
            I->first_err.compare_exchange_strong(z, -EIO);
        }
    }
    commit();
    I->completed.fetch_add(n, std::memory_order_release);
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
    cudaHostGetDevicePointer((void**)&I->area_d, I->area_h, 0);
    size_t inl = (size_t)slots * GSYS_INLINE_BYTES;
    if (cudaHostAlloc((void**)&I->inline_h, inl, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
        return fail(-ENOMEM);
    cudaHostGetDevicePointer((void**)&I->inline_d, I->inline_h, 0);
    if (cudaHostAlloc((void**)&I->ring_h, (size_t)rc * 8, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
        return fail(-ENOMEM);
    memset(I->ring_h, 0, (size_t)rc * 8);
    cudaHostGetDevicePointer((void**)&I->ring_d, I->ring_h, 0);
    if (cudaMalloc(&I->claim_d, (size_t)slots * 4) != cudaSuccess) return fail(-ENOMEM);
    if (cudaMalloc(&I->seqs_d, (size_t)slots * 4) != cudaSuccess) return fail(-ENOMEM);
    if (cudaMalloc(&I->mirror_d, (size_t)slots * 8) != cudaSuccess) return fail(-ENOMEM);
    if (cudaMalloc(&I->tail_d, 64) != cudaSuccess) return fail(-ENOMEM);
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
    cudaStreamCreateWithFlags(&I->ctl, cudaStreamNonBlocking);
    gsys_dev_ctx& c = I->ctx_h;
    c.area = I->area_d;
    c.inline_buf = I->inline_d;
    c.claim = I->claim_d;
    c.seqs = I->seqs_d;
    c.mirror = I->mirror_d;
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
    if (cudaMemcpy(I->ctx_d, &c, sizeof c, cudaMemcpyHostToDevice) != cudaSuccess) return fail(-EIO);
    if (cudaDeviceSynchronize() != cudaSuccess) return fail(-EIO);

    // service threads
    long cores = (long)std::thread::hardware_concurrency();
    cpu_set_t cs;
    if (sched_getaffinity(0, sizeof cs, &cs) == 0) cores = CPU_COUNT(&cs);
    uint32_t nthr = (uint32_t)std::max<long>(1, std::min<long>(12, cores / 2));
    ev = getenv("GSYS_THREADS");
    if (ev && atoi(ev) > 0) nthr = (uint32_t)atoi(ev);
    I->nthreads = nthr;
    size_t qcap = 1;
    while (qcap < (size_t)rc) qcap <<= 1;
    I->queue = new MPMC(qcap);
    size_t bcap = 32ull << 20;
    ev = getenv("GSYS_BOUNCE_MB");
    if (ev && atoi(ev) > 0) bcap = (size_t)atoi(ev) << 20;
    for (uint32_t t = 0; t < nthr; t++) {
        Worker* w = new Worker();
        w->inst = I;
        w->id = (int)t;
        cudaStreamCreateWithFlags(&w->stream, cudaStreamNonBlocking);
        if (cudaHostAlloc((void**)&w->bounce, bcap, cudaHostAllocDefault) != cudaSuccess) return fail(-ENOMEM);
        w->bcap = bcap;
        w->reqs.reserve(4096);
        w->ops.reserve(8192);
        I->workers.push_back(w);
    }
    for (Worker* w : I->workers) w->th = std::thread([w] { w->run(); });
    I->dispatcher = std::thread([I] { I->dispatch_loop(); });
    *out = I;
    return 0;
}

}  // namespace

// ====================================================================== internal API
gsys_dev_ctx* gsys_internal_ctx_d() {
    Instance* I = current();
    return I ? I->ctx_d : nullptr;
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

int gsys_launch(const void* kernel, uint32_t gx, uint32_t gy, uint32_t gz, uint32_t bx, uint32_t by, uint32_t bz,
                void** args, size_t smem_bytes, void* stream) {
    Instance* I = current();
    if (!I) return -ENODEV;
    if (!kernel || gx == 0 || gy == 0 || gz == 0 || bx == 0 || by == 0 || bz == 0) return -EINVAL;
    cudaStream_t s = (cudaStream_t)stream;
    uint64_t nb = (uint64_t)gx * gy * gz;
    if (nb > (1ull << 31)) return -EINVAL;
    if (nb > I->kblock_cap) {
        uint32_t cap = I->kblock_cap;
        while (cap < nb) cap <<= 1;
        uint32_t* nk = nullptr;
        if (cudaMalloc(&nk, (size_t)cap * GSYS_KSITES * 4) != cudaSuccess) return -ENOMEM;
        cudaStreamSynchronize(s);
        I->graveyard.push_back(I->kblock_d);
        I->kblock_d = nk;
        I->kblock_cap = cap;
        I->ctx_h.kblock = nk;
        I->ctx_h.kblock_cap = cap;
        if (cudaMemcpy(I->ctx_d, &I->ctx_h, sizeof I->ctx_h, cudaMemcpyHostToDevice) != cudaSuccess) return -EIO;
    }
    // reset the kernel-scope call sites for this launch (block rounds + per-round records)
    cudaMemsetAsync(I->kblock_d, 0, (size_t)nb * GSYS_KSITES * 4, s);
    cudaMemsetAsync(I->krounds_d, 0, sizeof(gsys_kround) * GSYS_KSITES * GSYS_KROUNDS, s);
    I->gen.fetch_add(1);
    I->kick.fetch_add(1);
    cudaError_t e = cudaLaunchKernel(kernel, dim3(gx, gy, gz), dim3(bx, by, bz), args, smem_bytes, s);
    return cuda_err(e);
}

int gsys_wait(void* stream) {
    Instance* I = current();
    if (!I) return -ENODEV;
    cudaError_t e = stream ? cudaStreamSynchronize((cudaStream_t)stream) : cudaDeviceSynchronize();
    if (e != cudaSuccess) return cuda_err(e);
    uint32_t tail = 0;
    cudaMemcpyAsync(&tail, I->tail_d, 4, cudaMemcpyDeviceToHost, I->ctl);
    cudaStreamSynchronize(I->ctl);
    uint64_t h = I->head.load(std::memory_order_acquire);
    uint64_t issued = h + (uint64_t)(uint32_t)(tail - (uint32_t)h);
    while (I->head.load(std::memory_order_acquire) < issued || I->completed.load(std::memory_order_acquire) < issued)
        std::this_thread::yield();
    for (Worker* w : I->workers) cudaStreamSynchronize(w->stream);
    return I->first_err.exchange(0);
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
    if (I->dispatcher.joinable()) I->dispatcher.join();
    for (Worker* w : I->workers) {
        if (w->th.joinable()) w->th.join();
        cudaStreamSynchronize(w->stream);
        for (auto& rg : w->inflight) if (rg.ev && rg.last) cudaEventDestroy(rg.ev);
        for (auto e : w->evpool) cudaEventDestroy(e);
        cudaStreamDestroy(w->stream);
        cudaFreeHost(w->bounce);
        delete w;
    }
    delete I->queue;
    cudaFreeHost(I->area_h);
    cudaFreeHost(I->inline_h);
    cudaFreeHost(I->ring_h);
    cudaFree(I->claim_d);
    cudaFree(I->seqs_d);
    cudaFree(I->mirror_d);
    cudaFree(I->tail_d);
    cudaFree(I->krounds_d);
    cudaFree(I->kblock_d);
    cudaFree(I->ctx_d);
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
    out->threads = I->nthreads;
    out->slots = I->nslots;
    out->coalesce_max = I->coalesce_max.load();
    out->coalesce_window_us = I->window_us.load();
    return 0;
}

int gsys_stats_reset(void) {
    Instance* I = current();
    if (!I) return -ENODEV;
    I->st_bundles.store(0);
    I->st_max_bundle.store(0);
    I->st_host_preads.store(0);
    I->st_merged.store(0);
    I->st_bytes_read.store(0);
    I->st_bytes_h2d.store(0);
    I->st_errors.store(0);
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

int64_t gsys_split_result(int64_t r, uint64_t offset_in_group, uint64_t len) {
    if (r < 0) return r;
    int64_t v = r - (int64_t)offset_in_group;
    if (v < 0) v = 0;
    if ((uint64_t)v > len) v = (int64_t)len;
    return v;
}

}  // extern "C"
