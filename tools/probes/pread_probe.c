// pread_probe.c -- host-side ceiling of the wordcount's data path: T threads issue pread(2) of
// `chunk` bytes from the corpus files into `nlines` distinct lines of a caller-supplied (pinned)
// buffer, round-robin over the corpus, for `secs` seconds.  Returns bytes/s.  Diagnostic only.
#define _GNU_SOURCE
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <time.h>
#include <unistd.h>

typedef struct {
    const int* fds; int nfiles; uint64_t fsize; uint8_t* buf; uint64_t chunk; int nlines;
    int tid, nthreads; volatile int* stop; uint64_t bytes;
} Arg;

static void* worker(void* p) {
    Arg* a = (Arg*)p;
    const uint64_t per_file = a->fsize / a->chunk;
    uint64_t k = a->tid;
    while (!*a->stop) {
        const uint64_t f = (k / per_file) % a->nfiles, c = k % per_file;
        uint8_t* dst = a->buf + (k % a->nlines) * a->chunk;
        ssize_t r = pread(a->fds[f], dst, a->chunk, c * a->chunk);
        if (r > 0) a->bytes += (uint64_t)r;
        k += a->nthreads;
    }
    return 0;
}

double pread_probe(const int* fds, int nfiles, uint64_t fsize, uint8_t* buf, uint64_t chunk, int nlines,
                   int nthreads, double secs) {
    pthread_t th[256];
    Arg args[256];
    volatile int stop = 0;
    struct timespec t0, t1;
    if (nthreads > 256) nthreads = 256;
    clock_gettime(CLOCK_MONOTONIC, &t0);
    for (int i = 0; i < nthreads; i++) {
        Arg a = {fds, nfiles, fsize, buf, chunk, nlines, i, nthreads, &stop, 0};
        args[i] = a;
        pthread_create(&th[i], 0, worker, &args[i]);
    }
    usleep((useconds_t)(secs * 1e6));
    stop = 1;
    uint64_t tot = 0;
    for (int i = 0; i < nthreads; i++) { pthread_join(th[i], 0); tot += args[i].bytes; }
    clock_gettime(CLOCK_MONOTONIC, &t1);
    return tot / ((t1.tv_sec - t0.tv_sec) + 1e-9 * (t1.tv_nsec - t0.tv_nsec));
}
