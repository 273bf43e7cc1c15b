/*
 * mc_client.c -- UDP load generator for the memcached-style workload (config 4).  Input side only:
 * it sends pre-encoded request packets and records each reply (matched by the opaque field) and
 * its round-trip latency.  Each of T threads owns one connected UDP socket and keeps at most
 * `window` requests in flight, so loopback buffers never overflow (no loss by construction; a
 * reply that does not arrive within the timeout is recorded as missing).
 */
#define _GNU_SOURCE
#include <arpa/inet.h>
#include <errno.h>
#include <netinet/in.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <sys/socket.h>
#include <time.h>
#include <unistd.h>

#define OPAQUE_BASE 0x10000000u

static uint64_t now_ns(void) {
    struct timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
}

typedef struct {
    int port, tid, nthreads, window;
    const uint8_t* pkts; const uint32_t* off; const uint32_t* len; uint32_t n;
    uint8_t* resp; uint32_t stride; uint32_t* rlen; uint64_t* lat; uint64_t* t_send;
    double timeout_s;
    int err;
} job_t;

static void* worker(void* arg) {
    job_t* J = (job_t*)arg;
    int fd = socket(AF_INET, SOCK_DGRAM, 0);
    if (fd < 0) { J->err = -errno; return NULL; }
    int rb = 8 << 20;
    setsockopt(fd, SOL_SOCKET, SO_RCVBUF, &rb, sizeof rb);
    struct timeval tv = {0, 200000};
    setsockopt(fd, SOL_SOCKET, SO_RCVTIMEO, &tv, sizeof tv);
    struct sockaddr_in sa;
    memset(&sa, 0, sizeof sa);
    sa.sin_family = AF_INET;
    sa.sin_port = htons((uint16_t)J->port);
    sa.sin_addr.s_addr = htonl(0x7f000001);
    if (connect(fd, (struct sockaddr*)&sa, sizeof sa) != 0) { J->err = -errno; close(fd); return NULL; }
    uint8_t buf[8192];
    uint32_t next = (uint32_t)J->tid, inflight = 0, done = 0, mine = 0;
    for (uint32_t i = (uint32_t)J->tid; i < J->n; i += (uint32_t)J->nthreads) mine++;
    uint64_t deadline = now_ns() + (uint64_t)(J->timeout_s * 1e9);
    while (done < mine && now_ns() < deadline) {
        while (inflight < (uint32_t)J->window && next < J->n) {
            J->t_send[next] = now_ns();
            if (send(fd, J->pkts + J->off[next], J->len[next], 0) < 0) { J->err = -errno; break; }
            next += (uint32_t)J->nthreads;
            inflight++;
        }
        ssize_t r = recv(fd, buf, sizeof buf, 0);
        if (r < 0) {
            if (errno == EAGAIN || errno == EWOULDBLOCK || errno == EINTR) {
                if (inflight && next >= J->n) { done += inflight; inflight = 0; }   /* give up on lost ones */
                continue;
            }
            J->err = -errno;
            break;
        }
        if (r < 32) continue;
        uint32_t opq = ((uint32_t)buf[20] << 24) | ((uint32_t)buf[21] << 16) | ((uint32_t)buf[22] << 8) | buf[23];
        if (opq < OPAQUE_BASE || opq - OPAQUE_BASE >= J->n) continue;
        uint32_t idx = opq - OPAQUE_BASE;
        if (J->rlen[idx] == 0) {
            uint32_t k = (uint32_t)r < J->stride ? (uint32_t)r : J->stride;
            memcpy(J->resp + (size_t)idx * J->stride, buf, k);
            J->rlen[idx] = k;
            J->lat[idx] = now_ns() - J->t_send[idx];
            done++;
            if (inflight) inflight--;
        }
    }
    close(fd);
    return NULL;
}

int mc_client_run(int port, const uint8_t* pkts, const uint32_t* off, const uint32_t* len, uint32_t n, int nthreads,
                  int window, uint8_t* resp, uint32_t stride, uint32_t* rlen, uint64_t* lat, double timeout_s,
                  double* secs) {
    if (nthreads < 1 || window < 1) return -EINVAL;
    uint64_t* t_send = (uint64_t*)calloc(n ? n : 1, sizeof(uint64_t));
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * nthreads);
    job_t* J = (job_t*)calloc(nthreads, sizeof(job_t));
    uint64_t t0 = now_ns();
    for (int t = 0; t < nthreads; t++) {
        job_t j = {port, t, nthreads, window, pkts, off, len, n, resp, stride, rlen, lat, t_send, timeout_s, 0};
        J[t] = j;
        pthread_create(&th[t], NULL, worker, &J[t]);
    }
    int err = 0;
    for (int t = 0; t < nthreads; t++) {
        pthread_join(th[t], NULL);
        if (J[t].err && !err) err = J[t].err;
    }
    if (secs) *secs = (now_ns() - t0) * 1e-9;
    free(t_send); free(th); free(J);
    return err;
}
