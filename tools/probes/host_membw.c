// Host memory bandwidth of the GPU box: T threads each memcpy a private 256 MiB buffer repeatedly;
// reports bytes moved (read + write) per second.  The wordcount moves ~3 host bytes per corpus
// byte (page cache -> bounce by pread, bounce -> GPU over PCIe), so this bounds it from the host side.
// gcc -O2 -pthread -o /tmp/host_membw host_membw.c && /tmp/host_membw 16
#include <pthread.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>

static size_t N = 256u << 20;
static double secs = 2.0;
static double now(void) { struct timespec t; clock_gettime(CLOCK_MONOTONIC, &t); return t.tv_sec + t.tv_nsec * 1e-9; }
typedef struct { double bytes; } Res;
static void* run(void* arg) {
    Res* r = (Res*)arg;
    char* a = malloc(N); char* b = malloc(N);
    memset(a, 1, N); memset(b, 2, N);
    double t0 = now(); r->bytes = 0;
    while (now() - t0 < secs) {
        memcpy(b, a, N);
        __asm__ volatile("" : : "r"(b), "r"(a) : "memory");   /* keep the copy */
        r->bytes += 2.0 * N;
    }
    if (b[N / 2] != 1) fprintf(stderr, "copy check failed\n");
    r->bytes /= (now() - t0);
    free(a); free(b);
    return NULL;
}
int main(int argc, char** argv) {
    int maxt = argc > 1 ? atoi(argv[1]) : 16;
    for (int t = 1; t <= maxt; t *= 2) {
        pthread_t th[256]; Res r[256];
        for (int i = 0; i < t; i++) pthread_create(&th[i], NULL, run, &r[i]);
        double tot = 0;
        for (int i = 0; i < t; i++) { pthread_join(th[i], NULL); tot += r[i].bytes; }
        printf("{\"probe\": \"host_memcpy\", \"threads\": %d, \"GBps_read_plus_write\": %.1f}\n", t, tot / 1e9);
        fflush(stdout);
    }
    return 0;
}
