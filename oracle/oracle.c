/*
 * oracle.c -- CPU ORACLE for the GENESYS hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg may
 * load this library.  It shares no code, header, table or constant with the CUDA path
 * (paper_conf_isca_veselybblor18_b200/ and include/), and never imports it.
 *
 * What it computes, each function citing the passage it follows (PAPER.md line + section):
 *   - oracle_pread / oracle_exec_plan: "the same syscalls directly from host threads"
 *     (BASELINE.json north_star) -- plain libc pread(2), the call GENESYS forwards with
 *     "standard POSIX semantics" (sec. I, P10.23).  Raw convention: >=0 or -errno.
 *   - oracle_count_tokens: wordcount, "search for occurrences of 64 strings" (PAPER.md:32
 *     sec. VIII-C, P32.6).  Reading A9: a token is a maximal run of [A-Za-z0-9_],
 *     a hit is a whole token byte-equal to a dictionary word (case-sensitive ASCII).
 *     Written as the plain definition: a scalar byte loop over the whole file.
 *   - oracle_grep: grep -F -l, "identifying which files contain any of the words on the list"
 *     (sec. VIII-C, P30.28); substring test, stops at the first hit (P30.38).
 *   - oracle_corpus: both over a list of files, files split across T pthreads (the paper's
 *     OpenMP CPU version, P32.8), each file read with the same chunked pread plan
 *     the GPU work-groups issue (one pread per work-group chunk, PAPER.md:32 P32.7).
 *   - oracle_getrusage_rate / oracle_pread_rate: direct host syscall rates for the
 *     granularity microbenchmark baseline (sec. VII, P26.5-16).
 */
#define _GNU_SOURCE
#include <errno.h>
#include <fcntl.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <sys/resource.h>
#include <sys/socket.h>
#include <sys/stat.h>
#include <sys/types.h>
#include <time.h>
#include <unistd.h>

#define O_NDICT 64
#define O_DSTRIDE 17

static double now_s(void) {
    struct timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return ts.tv_sec + ts.tv_nsec * 1e-9;
}

/* pread(2) with the raw-syscall return convention (>= 0 bytes, or -errno). */
int64_t oracle_pread(int fd, void* buf, uint64_t n, int64_t off) {
    ssize_t r = pread(fd, buf, (size_t)n, (off_t)off);
    return r < 0 ? -(int64_t)errno : (int64_t)r;
}

/*
 * Execute a request plan: for each i, pread(fd[i], base + dst_off[i], len[i], off[i]), recording
 * the return in ret[i].  Requests run in plan order from one thread (results are per request id,
 * never by arrival order, reading A18).
 */
int oracle_exec_plan(int n, const int* fd, const int64_t* off, const uint64_t* len,
                     uint8_t* base, const uint64_t* dst_off, int64_t* ret) {
    for (int i = 0; i < n; i++) ret[i] = oracle_pread(fd[i], base + dst_off[i], len[i], off[i]);
    return 0;
}

static inline int is_word_byte(uint8_t c) {
    return (c >= 'a' && c <= 'z') || (c >= 'A' && c <= 'Z') || (c >= '0' && c <= '9') || c == '_';
}

/* Whole-token dictionary counts over text[0, n): hist[j] += #tokens equal to dict word j. */
void oracle_count_tokens(const uint8_t* text, uint64_t n, const char* dict, const uint8_t* dlen,
                         int ndict, uint64_t* hist) {
    uint64_t i = 0;
    while (i < n) {
        if (!is_word_byte(text[i])) { i++; continue; }
        uint64_t j = i;
        while (j < n && is_word_byte(text[j])) j++;
        uint64_t len = j - i;
        for (int d = 0; d < ndict; d++) {
            if (dlen[d] == len && memcmp(text + i, dict + O_DSTRIDE * d, len) == 0) { hist[d]++; break; }
        }
        i = j;
    }
}

/* 1 if any pattern occurs as a substring of text[0, n) (grep -F semantics), else 0. */
int oracle_grep(const uint8_t* text, uint64_t n, const char* pats, const uint8_t* plen, int npat) {
    for (uint64_t i = 0; i < n; i++) {
        for (int p = 0; p < npat; p++) {
            uint64_t L = plen[p];
            if (L && i + L <= n && memcmp(text + i, pats + O_DSTRIDE * p, L) == 0) return 1;
        }
    }
    return 0;
}

/*
 * Read a whole file through the work-group pread plan: chunk c covers [c*chunk, (c+1)*chunk);
 * its request is pread(off = max(s-1, 0), len = (e+16) - off) where e = min(s+chunk, size) --
 * the GPU work-group's halo request (reading A10).  Bytes [s, e) of each reply are placed at
 * out[s..e).  Returns 0, or -errno of the first failed pread, or -EIO on a short read that
 * does not cover [s, e).
 */
int oracle_read_file_plan(int fd, uint64_t size, uint64_t chunk, uint8_t* out, uint8_t* scratch,
                          int64_t* rets) {
    uint64_t nch = (size + chunk - 1) / chunk;
    for (uint64_t c = 0; c < nch; c++) {
        uint64_t s = c * chunk, e = s + chunk < size ? s + chunk : size;
        uint64_t off = s ? s - 1 : 0;
        uint64_t len = e + 16 - off;
        int64_t r = oracle_pread(fd, scratch, len, (int64_t)off);
        if (rets) rets[c] = r;
        if (r < 0) return (int)r;
        if ((uint64_t)r < e - off) return -EIO;
        memcpy(out + s, scratch + (s - off), e - s);
    }
    return 0;
}

typedef struct {
    const char* const* paths;
    int nfiles;
    uint64_t chunk;
    const char* dict; const uint8_t* dlen; int ndict;
    const char* pats; const uint8_t* plen; int npat;
    int next;
    pthread_mutex_t mu;
    uint64_t hist[O_NDICT];
    uint32_t* file_hits;
    uint64_t bytes;
    int err;
} corpus_job_t;

static void* corpus_worker(void* arg) {
    corpus_job_t* J = (corpus_job_t*)arg;
    uint64_t hist[O_NDICT];
    memset(hist, 0, sizeof hist);
    uint64_t bytes = 0;
    uint8_t* scratch = (uint8_t*)malloc(J->chunk + 64);
    uint8_t* buf = NULL;
    uint64_t cap = 0;
    int err = 0;
    for (;;) {
        pthread_mutex_lock(&J->mu);
        int f = J->next++;
        pthread_mutex_unlock(&J->mu);
        if (f >= J->nfiles) break;
        int fd = open(J->paths[f], O_RDONLY);
        if (fd < 0) { err = -errno; continue; }
        struct stat st;
        if (fstat(fd, &st) != 0) { err = -errno; close(fd); continue; }
        uint64_t size = (uint64_t)st.st_size;
        if (size > cap) { free(buf); cap = size; buf = (uint8_t*)malloc(cap ? cap : 1); }
        int r = oracle_read_file_plan(fd, size, J->chunk, buf, scratch, NULL);
        close(fd);
        if (r) { err = r; continue; }
        oracle_count_tokens(buf, size, J->dict, J->dlen, J->ndict, hist);
        if (J->file_hits) J->file_hits[f] = (uint32_t)oracle_grep(buf, size, J->pats, J->plen, J->npat);
        bytes += size;
    }
    free(buf);
    free(scratch);
    pthread_mutex_lock(&J->mu);
    for (int d = 0; d < O_NDICT; d++) J->hist[d] += hist[d];
    J->bytes += bytes;
    if (err && !J->err) J->err = err;
    pthread_mutex_unlock(&J->mu);
    return NULL;
}

/*
 * Wordcount + grep -F -l over nfiles files with nthreads host threads.  hist[64] is overwritten;
 * file_hits[f] (may be NULL) = 1 if file f contains any pattern.  *secs = wall time.
 * Returns 0 or the first -errno.
 */
int oracle_corpus(const char* const* paths, int nfiles, int nthreads, uint64_t chunk,
                  const char* dict, const uint8_t* dlen, int ndict,
                  const char* pats, const uint8_t* plen, int npat,
                  uint64_t* hist, uint32_t* file_hits, double* secs) {
    if (ndict > O_NDICT || nthreads < 1 || chunk == 0) return -EINVAL;
    corpus_job_t J;
    memset(&J, 0, sizeof J);
    J.paths = paths; J.nfiles = nfiles; J.chunk = chunk;
    J.dict = dict; J.dlen = dlen; J.ndict = ndict;
    J.pats = pats; J.plen = plen; J.npat = npat;
    J.file_hits = file_hits;
    pthread_mutex_init(&J.mu, NULL);
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * nthreads);
    double t0 = now_s();
    for (int t = 0; t < nthreads; t++) pthread_create(&th[t], NULL, corpus_worker, &J);
    for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
    double t1 = now_s();
    free(th);
    pthread_mutex_destroy(&J.mu);
    for (int d = 0; d < ndict; d++) hist[d] = J.hist[d];
    if (secs) *secs = t1 - t0;
    return J.err;
}

/* Occurrences (overlapping) of key[0..k) in data[0..n): the signal-search lookup of PAPER.md:30
 * sec. VIII-B ("parallel lookup in a data array"), written as the definition. */
uint64_t oracle_count_key(const uint8_t* data, uint64_t n, const uint8_t* key, uint64_t k) {
    uint64_t c = 0;
    if (k == 0 || k > n) return 0;
    for (uint64_t i = 0; i + k <= n; i++)
        if (memcmp(data + i, key, k) == 0) c++;
    return c;
}

typedef struct {
    const char* const* paths; int nfiles; uint64_t chunk; int next; pthread_mutex_t mu; uint64_t bytes; int err;
} pread_job_t;

static void* pread_only_worker(void* arg) {
    pread_job_t* J = (pread_job_t*)arg;
    uint8_t* buf = (uint8_t*)malloc(J->chunk + 64);
    uint64_t bytes = 0;
    int err = 0;
    for (;;) {
        pthread_mutex_lock(&J->mu);
        int f = J->next++;
        pthread_mutex_unlock(&J->mu);
        if (f >= J->nfiles) break;
        int fd = open(J->paths[f], O_RDONLY);
        if (fd < 0) { err = -errno; continue; }
        for (uint64_t off = 0;; off += J->chunk) {
            ssize_t r = pread(fd, buf, J->chunk, (off_t)off);
            if (r < 0) { err = -errno; break; }
            bytes += (uint64_t)r;
            if ((uint64_t)r < J->chunk) break;
        }
        close(fd);
    }
    free(buf);
    pthread_mutex_lock(&J->mu);
    J->bytes += bytes;
    if (err && !J->err) J->err = err;
    pthread_mutex_unlock(&J->mu);
    return NULL;
}

/* Host pread ceiling: nthreads threads pread every file in `chunk`-byte calls into private
 * buffers, no scan (the host-side co-roofline of the GPU-syscall wordcount).  Returns bytes/s
 * (or a negative errno). */
double oracle_pread_only(const char* const* paths, int nfiles, int nthreads, uint64_t chunk) {
    pread_job_t J;
    memset(&J, 0, sizeof J);
    J.paths = paths; J.nfiles = nfiles; J.chunk = chunk;
    pthread_mutex_init(&J.mu, NULL);
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * nthreads);
    double t0 = now_s();
    for (int t = 0; t < nthreads; t++) pthread_create(&th[t], NULL, pread_only_worker, &J);
    for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
    double dt = now_s() - t0;
    free(th);
    pthread_mutex_destroy(&J.mu);
    if (J.err) return (double)J.err;
    return (double)J.bytes / dt;
}

typedef struct { uint64_t iters; int fd; uint64_t len; uint64_t size; int kind; int tid; int err; } rate_job_t;

static void* rate_worker(void* arg) {
    rate_job_t* R = (rate_job_t*)arg;
    if (R->kind == 0) {
        struct rusage ru;
        for (uint64_t i = 0; i < R->iters; i++)
            if (getrusage(RUSAGE_SELF, &ru) != 0) R->err = -errno;
    } else {
        uint8_t* b = (uint8_t*)malloc(R->len);
        uint64_t slots = R->size / R->len ? R->size / R->len : 1;
        for (uint64_t i = 0; i < R->iters; i++) {
            uint64_t off = ((i * 7919 + (uint64_t)R->tid * 104729) % slots) * R->len;
            if (pread(R->fd, b, R->len, (off_t)off) < 0) R->err = -errno;
        }
        free(b);
    }
    return NULL;
}

/* Direct host syscall rate (calls/s) with nthreads threads: kind 0 = getrusage(RUSAGE_SELF)
 * (144 B struct out), kind 1 = pread(fd, len) at rotating aligned offsets of a size-byte file. */
double oracle_syscall_rate(int kind, int nthreads, uint64_t iters_per_thread, int fd, uint64_t len,
                           uint64_t size) {
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * nthreads);
    rate_job_t* R = (rate_job_t*)calloc(nthreads, sizeof(rate_job_t));
    for (int t = 0; t < nthreads; t++) {
        R[t].iters = iters_per_thread; R[t].fd = fd; R[t].len = len; R[t].size = size;
        R[t].kind = kind; R[t].tid = t;
    }
    double t0 = now_s();
    for (int t = 0; t < nthreads; t++) pthread_create(&th[t], NULL, rate_worker, &R[t]);
    for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
    double dt = now_s() - t0;
    int err = 0;
    for (int t = 0; t < nthreads; t++) if (R[t].err) err = R[t].err;
    free(th); free(R);
    if (err) return (double)err;
    return (double)iters_per_thread * nthreads / dt;
}

/*
 * CPU memcached-style GET server (config 4 baseline, sec. VIII-D "a CPU version of this
 * workload"): nthreads threads loop recvfrom(fd) -> look the key up -> sendto, until *stop.  The
 * store is the plain list of n (key, value) pairs grouped into nbuckets buckets by a djb2 hash of
 * the key (the CPU version's own table; nothing is shared with the GPU path), scanned linearly.
 * Replies follow the definition in oracle/mc.py.  Returns requests served.
 */
typedef struct {
    int fd; volatile int* stop;
    const uint8_t* keys; const uint32_t* koff; const uint8_t* klen;
    const uint8_t* vals; const uint64_t* voff; const uint32_t* vlen;
    const uint32_t* order; const uint32_t* bstart; uint32_t nbuckets;
    uint64_t served;
} mc_job_t;

static uint32_t djb2(const uint8_t* k, uint32_t n) {
    uint32_t h = 5381;
    for (uint32_t i = 0; i < n; i++) h = h * 33u + k[i];
    return h;
}

static void* mc_worker(void* arg) {
    mc_job_t* J = (mc_job_t*)arg;
    uint8_t rx[2048], tx[8192];
    uint64_t served = 0;
    while (!*J->stop) {
        struct sockaddr_storage from;
        socklen_t fl = sizeof from;
        ssize_t r = recvfrom(J->fd, rx, sizeof rx, 0, (struct sockaddr*)&from, &fl);
        if (r < 32 || rx[8] != 0x80 || rx[9] != 0x00) continue;
        uint32_t klen = ((uint32_t)rx[10] << 8) | rx[11], ext = rx[12];
        if (klen < 1 || klen > 32 || 32 + ext + klen > (uint32_t)r) continue;
        const uint8_t* key = rx + 32 + ext;
        uint32_t b = djb2(key, klen) % J->nbuckets;
        int64_t hit = -1;
        for (uint32_t j = J->bstart[b]; j < J->bstart[b + 1]; j++) {
            uint32_t i = J->order[j];
            if (J->klen[i] == klen && memcmp(J->keys + J->koff[i], key, klen) == 0) { hit = i; break; }
        }
        memset(tx, 0, 36);
        tx[0] = rx[0]; tx[1] = rx[1]; tx[5] = 1;
        tx[8] = 0x81; tx[9] = rx[9];
        uint32_t body = hit >= 0 ? 4 + J->vlen[hit] : 9;
        tx[12] = hit >= 0 ? 4 : 0;
        tx[15] = hit >= 0 ? 0 : 1;
        tx[16] = (uint8_t)(body >> 24); tx[17] = (uint8_t)(body >> 16); tx[18] = (uint8_t)(body >> 8); tx[19] = (uint8_t)body;
        memcpy(tx + 20, rx + 20, 4);
        size_t len;
        if (hit >= 0) { memcpy(tx + 36, J->vals + J->voff[hit], J->vlen[hit]); len = 36 + J->vlen[hit]; }
        else { memcpy(tx + 32, "Not found", 9); len = 41; }
        sendto(J->fd, tx, len, 0, (struct sockaddr*)&from, fl);
        served++;
    }
    __atomic_add_fetch(&J->served, served, __ATOMIC_RELAXED);
    return NULL;
}

int64_t oracle_mc_serve(int fd, int nthreads, const uint8_t* keys, const uint32_t* koff, const uint8_t* klen,
                        const uint8_t* vals, const uint64_t* voff, const uint32_t* vlen, uint32_t n,
                        uint32_t nbuckets, volatile int* stop) {
    uint32_t* bstart = (uint32_t*)calloc(nbuckets + 1, sizeof(uint32_t));
    uint32_t* order = (uint32_t*)malloc(sizeof(uint32_t) * (n ? n : 1));
    uint32_t* fill = (uint32_t*)calloc(nbuckets, sizeof(uint32_t));
    for (uint32_t i = 0; i < n; i++) bstart[djb2(keys + koff[i], klen[i]) % nbuckets + 1]++;
    for (uint32_t b = 0; b < nbuckets; b++) bstart[b + 1] += bstart[b];
    for (uint32_t i = 0; i < n; i++) {
        uint32_t b = djb2(keys + koff[i], klen[i]) % nbuckets;
        order[bstart[b] + fill[b]++] = i;
    }
    mc_job_t J = {fd, stop, keys, koff, klen, vals, voff, vlen, order, bstart, nbuckets, 0};
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * nthreads);
    for (int t = 0; t < nthreads; t++) pthread_create(&th[t], NULL, mc_worker, &J);
    for (int t = 0; t < nthreads; t++) pthread_join(th[t], NULL);
    free(th); free(bstart); free(order); free(fill);
    return (int64_t)J.served;
}
