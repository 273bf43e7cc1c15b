// Host memory-bandwidth hog for contention experiments: T threads memcpy private 256 MiB buffers
// until killed (emulates a GPU box whose host DRAM is shared with other work).  Prints the rate
// each thread saw once a second to stderr is skipped: the experiment measures the wordcount, not
// the hog.  gcc -O2 -pthread -o /tmp/membw_hog membw_hog.c && /tmp/membw_hog 3 &
#include <pthread.h>
#include <stdlib.h>
#include <string.h>

static const size_t N = 256u << 20;
static void* run(void* arg) {
    (void)arg;
    char* a = malloc(N);
    char* b = malloc(N);
    memset(a, 1, N);
    memset(b, 2, N);
    for (;;) {
        memcpy(b, a, N);
        __asm__ volatile("" : : "r"(b), "r"(a) : "memory");
    }
    return NULL;
}
int main(int argc, char** argv) {
    int t = argc > 1 ? atoi(argv[1]) : 2;
    pthread_t th[64];
    for (int i = 0; i < t && i < 64; i++) pthread_create(&th[i], NULL, run, NULL);
    pthread_join(th[0], NULL);
    return 0;
}
