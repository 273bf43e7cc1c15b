/*
 * gen_corpus.c -- seeded synthetic text generator shared by the oracle and the GPU path.
 *
 * INPUT CONSTRUCTION ONLY.  This file holds none of the method's arithmetic (no tokenizer, no
 * matcher, no pread planning); it writes bytes and records what it *inserted* (a census of the
 * dictionary words it emitted, and which grep patterns it planted in which file).  Both the
 * oracle (oracle/) and the CUDA path (paper_conf_isca_veselybblor18_b200/) read the same files.
 *
 * Workload shape follows the paper's storage workloads: wordcount "configured to search for
 * occurrences of 64 strings" (sec. VIII-C, P32.6) and grep -F -l over a list of
 * words and files (sec. VIII-C, P30.27-29).  The recipe:
 *   - vocabulary V = 32768 unique lowercase words, lengths 1..20 (mean ~5.3), Zipf(s=1.07);
 *   - separators: ' ' mostly, '\n' when the line passes a 60..100 byte target, ",.;:!?"+' ' (8%);
 *   - text is produced in independent 4 KiB blocks, keyed by (seed, file, block) through a
 *     counter-based splitmix64, so files are reproducible and generated in parallel;
 *   - every block holds whole tokens only (padding with ' '), so the only tokens in a file are
 *     vocabulary words, planted dictionary words and planted grep patterns;
 *   - boundary plants: at each 4 KiB multiple B (which includes every 64 KiB and 256 KiB
 *     boundary) with probability 1/2 a present dictionary word is written starting at B-3,
 *     i.e. straddling the boundary, to exercise chunk-boundary ownership;
 *   - grep plants (plant seed, ~25% of files): 1..3 standalone tokens drawn from 8 patterns of
 *     12..16 bytes that start with a digit and contain an uppercase letter -- characters the
 *     text never emits elsewhere, so the per-file grep answer is known by construction;
 *   - dictionary (64 words): ranks 1-16, 101-116, 1001-1014 + one 15 B and one 16 B word,
 *     8 absent words ('Z'+lowercase, never emitted), 4 proper prefixes and 4 proper suffixes of
 *     frequent words that are not in V (whole-token count 0 by construction).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

#define V_WORDS 32768
#define MAX_WLEN 20
#define NDICT 64
#define NPAT 8
#define BLOCK 4096

static inline uint64_t mix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

typedef struct { uint64_t s; } rng_t;
static inline uint64_t rng_next(rng_t* r) {
    r->s += 0x9E3779B97F4A7C15ull;
    uint64_t z = r->s;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
static inline rng_t rng_key(uint64_t a, uint64_t b, uint64_t c) {
    rng_t r; r.s = mix64(a ^ mix64(b ^ mix64(c ^ 0x5851F42D4C957F2Dull))); return r;
}

static char g_vocab[V_WORDS][MAX_WLEN + 1];
static uint8_t g_vlen[V_WORDS];
static double g_cdf[V_WORDS];
static int16_t g_dict_of_vocab[V_WORDS];     /* -1 or dictionary index */
static char g_dict[NDICT][17];
static uint8_t g_dlen[NDICT];
static char g_pat[NPAT][17];
static uint8_t g_plen[NPAT];
static int g_ready = 0;
static uint64_t g_dict_seed = 0;

/* per-mille length weights for lengths 1..20 */
static const int k_len_w[MAX_WLEN] = {30,100,150,160,140,110,90,70,50,35,22,14,10,7,4,3,2,1,1,1};

/* simple open-addressing set of vocab strings for uniqueness checks */
#define HSET (1 << 17)
static int32_t g_hset[HSET];
static uint64_t str_hash(const char* s, int n) {
    uint64_t h = 1469598103934665603ull;
    for (int i = 0; i < n; i++) { h ^= (uint8_t)s[i]; h *= 1099511628211ull; }
    return mix64(h);
}
static int vocab_find(const char* s, int n) {
    uint64_t h = str_hash(s, n) & (HSET - 1);
    while (g_hset[h] >= 0) {
        int i = g_hset[h];
        if (g_vlen[i] == n && memcmp(g_vocab[i], s, n) == 0) return i;
        h = (h + 1) & (HSET - 1);
    }
    return -1;
}
static void vocab_insert(int idx) {
    uint64_t h = str_hash(g_vocab[idx], g_vlen[idx]) & (HSET - 1);
    while (g_hset[h] >= 0) h = (h + 1) & (HSET - 1);
    g_hset[h] = idx;
}
static int dict_has(int upto, const char* s, int n) {
    for (int j = 0; j < upto; j++)
        if (g_dlen[j] == n && memcmp(g_dict[j], s, n) == 0) return 1;
    return 0;
}

int gen_init(uint64_t dict_seed) {
    if (g_ready && g_dict_seed == dict_seed) return 0;
    memset(g_hset, 0xff, sizeof(g_hset));
    rng_t r = rng_key(dict_seed, 0xC0FFEEull, 1);
    for (int i = 0; i < V_WORDS; i++) {
        for (;;) {
            int u = (int)(rng_next(&r) % 1000), L = 0, acc = 0;
            while (L < MAX_WLEN) { acc += k_len_w[L]; L++; if (u < acc) break; }
            for (int k = 0; k < L; k++) g_vocab[i][k] = (char)('a' + rng_next(&r) % 26);
            g_vocab[i][L] = 0;
            g_vlen[i] = (uint8_t)L;
            if (vocab_find(g_vocab[i], L) < 0) break;
        }
        vocab_insert(i);
    }
    /* Zipf(s=1.07) cumulative distribution over ranks 1..V */
    double z = 0;
    for (int i = 0; i < V_WORDS; i++) z += pow((double)(i + 1), -1.07);
    double acc = 0;
    for (int i = 0; i < V_WORDS; i++) { acc += pow((double)(i + 1), -1.07) / z; g_cdf[i] = acc; }
    g_cdf[V_WORDS - 1] = 1.0;

    /* dictionary */
    int d = 0;
    for (int i = 0; i < 16; i++, d++) { memcpy(g_dict[d], g_vocab[i], 17); g_dlen[d] = g_vlen[i] > 16 ? 16 : g_vlen[i]; }
    for (int i = 100; i < 116; i++, d++) { memcpy(g_dict[d], g_vocab[i], 17); g_dlen[d] = g_vlen[i]; }
    for (int i = 1000; i < 1014; i++, d++) { memcpy(g_dict[d], g_vocab[i], 17); g_dlen[d] = g_vlen[i]; }
    for (int want = 15; want <= 16; want++) {
        int pick = -1;
        for (int i = 1014; i < V_WORDS && pick < 0; i++) if (g_vlen[i] == want) pick = i;
        if (pick < 0) pick = 1014 + (want - 15);
        memcpy(g_dict[d], g_vocab[pick], 17); g_dlen[d] = g_vlen[pick]; d++;
    }
    /* words longer than 16 bytes cannot be dictionary words (<= 16 B): clip guard */
    for (int j = 0; j < d; j++) if (g_dlen[j] > 16) { g_dlen[j] = 16; g_dict[j][16] = 0; }
    {   /* absent: 'Z' + lowercase, never emitted (text has no uppercase outside grep plants,
           which are whole tokens starting with a digit) */
        static const int alen[8] = {3, 5, 7, 9, 11, 13, 15, 16};
        for (int k = 0; k < 8; k++, d++) {
            g_dict[d][0] = 'Z';
            for (int q = 1; q < alen[k]; q++) g_dict[d][q] = (char)('a' + rng_next(&r) % 26);
            g_dict[d][alen[k]] = 0; g_dlen[d] = (uint8_t)alen[k];
        }
    }
    {   /* adversarial proper prefixes / suffixes of frequent words, not in V */
        int got = 0;
        for (int i = 0; i < 2000 && got < 4; i++) {
            int L = g_vlen[i];
            if (L < 3 || L - 1 > 16) continue;
            int pl = L - 1;
            if (vocab_find(g_vocab[i], pl) >= 0 || dict_has(d, g_vocab[i], pl)) continue;
            memcpy(g_dict[d], g_vocab[i], pl); g_dict[d][pl] = 0; g_dlen[d] = (uint8_t)pl; d++; got++;
        }
        got = 0;
        for (int i = 0; i < 2000 && got < 4; i++) {
            int L = g_vlen[i];
            if (L < 3 || L - 1 > 16) continue;
            int sl = L - 1;
            const char* s = g_vocab[i] + 1;
            if (vocab_find(s, sl) >= 0 || dict_has(d, s, sl)) continue;
            memcpy(g_dict[d], s, sl); g_dict[d][sl] = 0; g_dlen[d] = (uint8_t)sl; d++; got++;
        }
    }
    if (d != NDICT) return -1;
    for (int j = 0; j < NDICT; j++)
        if (dict_has(j, g_dict[j], g_dlen[j])) return -2;   /* dictionary entries are unique */
    for (int i = 0; i < V_WORDS; i++) g_dict_of_vocab[i] = -1;
    for (int j = 0; j < NDICT; j++) {
        int v = vocab_find(g_dict[j], g_dlen[j]);
        if (v >= 0) g_dict_of_vocab[v] = (int16_t)j;
    }
    /* grep patterns: 12..16 bytes, first byte a digit, at least one uppercase */
    rng_t rp = rng_key(dict_seed, 0xBEEFull, 7);
    for (int p = 0; p < NPAT; p++) {
        int L = 12 + (int)(rng_next(&rp) % 5);
        static const char alpha[] = "ABCDEFGHIJKLMNOPQRSTUVWXYZ0123456789abcdefghijklmnopqrstuvwxyz";
        g_pat[p][0] = (char)('0' + rng_next(&rp) % 10);
        for (int k = 1; k < L; k++) g_pat[p][k] = alpha[rng_next(&rp) % 62];
        g_pat[p][1 + (int)(rng_next(&rp) % (L - 1))] = (char)('A' + rng_next(&rp) % 26);
        g_pat[p][L] = 0; g_plen[p] = (uint8_t)L;
    }
    g_ready = 1;
    g_dict_seed = dict_seed;
    return 0;
}

int gen_dict(char* out, uint8_t* lens) {
    if (!g_ready) return -1;
    for (int j = 0; j < NDICT; j++) { memcpy(out + 17 * j, g_dict[j], 17); lens[j] = g_dlen[j]; }
    return 0;
}
int gen_patterns(char* out, uint8_t* lens) {
    if (!g_ready) return -1;
    for (int p = 0; p < NPAT; p++) { memcpy(out + 17 * p, g_pat[p], 17); lens[p] = g_plen[p]; }
    return 0;
}
/* vocabulary rank of a dictionary word, -1 if it is not a vocabulary word */
int gen_dict_rank(int j) {
    if (!g_ready || j < 0 || j >= NDICT) return -2;
    return vocab_find(g_dict[j], g_dlen[j]);
}

static inline int zipf_draw(rng_t* r) {
    double u = (double)(rng_next(r) >> 11) * (1.0 / 9007199254740992.0);
    int lo = 0, hi = V_WORDS - 1;
    while (lo < hi) { int mid = (lo + hi) >> 1; if (g_cdf[mid] > u) hi = mid; else lo = mid + 1; }
    return lo;
}

/* Boundary plant at 4 KiB multiple B of a file of `size` bytes: returns dict index or -1. */
static int boundary_plant(uint64_t seed, uint64_t file_id, uint64_t B, uint64_t size) {
    if (B == 0 || B % BLOCK) return -1;
    uint64_t h = mix64(seed ^ mix64(file_id * 0xD6E8FEB86659FD93ull ^ mix64(B)));
    if (!(h & 1)) return -1;
    int w = (int)((h >> 8) % 48);                     /* present words only */
    if (B - 4 + (uint64_t)g_dlen[w] + 2 > size) return -1;   /* ' ' word ' ' must fit */
    return w;
}

typedef struct { int nplant; uint32_t blk[3]; uint16_t off[3]; uint8_t pat[3]; } grep_plan_t;

static void grep_plan(uint64_t plant_seed, uint64_t file_id, uint64_t size, grep_plan_t* gp) {
    gp->nplant = 0;
    uint64_t nfull = size / BLOCK;
    if (nfull < 4) return;
    rng_t r = rng_key(plant_seed, file_id, 0x6E7Bull);
    if (rng_next(&r) % 4 != 0) return;
    int n = 1 + (int)(rng_next(&r) % 3);
    for (int k = 0; k < n; k++) {
        uint32_t b;
        int again;
        do {
            b = (uint32_t)(rng_next(&r) % nfull);
            again = 0;
            for (int q = 0; q < k; q++) if (gp->blk[q] == b) again = 1;
        } while (again);
        gp->blk[k] = b;
        gp->off[k] = (uint16_t)(1024 + rng_next(&r) % 1024);
        gp->pat[k] = (uint8_t)(rng_next(&r) % NPAT);
    }
    gp->nplant = n;
}

/* Fill free range [a, b) of block-local buffer with whole tokens + separators, padding ' '. */
static void fill_range(uint8_t* blk, int a, int b, rng_t* r, int* line_len, int* line_tgt,
                       uint64_t* census) {
    int pos = a;
    for (;;) {
        int w = zipf_draw(r);
        int L = g_vlen[w];
        /* separator choice */
        uint64_t sr = rng_next(r);
        int punct = (sr % 100) < 8;
        int need = L + (punct ? 2 : 1);
        if (pos + need > b) break;
        memcpy(blk + pos, g_vocab[w], L);
        pos += L;
        if (census && g_dict_of_vocab[w] >= 0) census[g_dict_of_vocab[w]]++;
        *line_len += need;
        if (punct) { static const char pc[] = ",.;:!?"; blk[pos++] = (uint8_t)pc[(sr >> 8) % 6]; }
        if (*line_len >= *line_tgt) {
            blk[pos++] = '\n';
            *line_len = 0;
            *line_tgt = 60 + (int)((sr >> 16) % 41);
        } else {
            blk[pos++] = ' ';
        }
    }
    while (pos < b) blk[pos++] = ' ';
}

/*
 * Generate one file of `size` bytes into buf.  census[64] (may be NULL) is INCREMENTED by the
 * number of whole-token emissions of each dictionary word; *pmask receives the bitmask of grep
 * patterns planted in this file (0 when grep_plants == 0).
 */
int gen_file(uint64_t seed, uint64_t file_id, uint64_t plant_seed, int grep_plants,
             uint8_t* buf, uint64_t size, uint64_t* census, uint32_t* pmask) {
    if (!g_ready) return -1;
    grep_plan_t gp; gp.nplant = 0;
    if (grep_plants) grep_plan(plant_seed, file_id, size, &gp);
    uint32_t mask = 0;
    uint64_t nblk = (size + BLOCK - 1) / BLOCK;
    for (uint64_t bi = 0; bi < nblk; bi++) {
        uint64_t boff = bi * BLOCK;
        int bsz = (int)((size - boff) < BLOCK ? (size - boff) : BLOCK);
        uint8_t* blk = buf + boff;
        rng_t r = rng_key(seed, file_id, bi);
        int line_len = 0, line_tgt = 60 + (int)(rng_next(&r) % 41);
        /* reserved region at the start: tail of the plant straddling boundary boff */
        int a = 0;
        int ws = boundary_plant(seed, file_id, boff, size);
        if (ws >= 0) {
            /* plant bytes: ' ' at boff-4, word at boff-3.., ' ' at boff-3+len */
            int end_local = -3 + (int)g_dlen[ws] + 1;   /* exclusive end, block-local */
            a = end_local > 0 ? end_local : 0;
        }
        /* reserved region at the end: head of the plant straddling boundary boff+BLOCK */
        int b = bsz;
        int we = (bsz == BLOCK) ? boundary_plant(seed, file_id, boff + BLOCK, size) : -1;
        if (we >= 0) b = BLOCK - 4;
        /* grep plant inside this block */
        int gk = -1;
        for (int k = 0; k < gp.nplant; k++) if (gp.blk[k] == bi && bsz == BLOCK) gk = k;
        if (gk >= 0) {
            int o = gp.off[gk], pl = g_plen[gp.pat[gk]];
            if (o > a && o + pl + 2 <= b) {
                fill_range(blk, a, o, &r, &line_len, &line_tgt, census);
                blk[o] = ' ';
                memcpy(blk + o + 1, g_pat[gp.pat[gk]], pl);
                blk[o + 1 + pl] = ' ';
                mask |= 1u << gp.pat[gk];
                a = o + pl + 2;
            }
        }
        fill_range(blk, a, b, &r, &line_len, &line_tgt, census);
        if (we >= 0) {
            /* write the part of the straddling plant that lies in this block */
            blk[BLOCK - 4] = ' ';
            for (int q = 0; q < 3; q++) {
                int idx = q;                         /* word byte q at local BLOCK-3+q */
                if (idx < g_dlen[we]) blk[BLOCK - 3 + q] = (uint8_t)g_dict[we][idx];
                else if (idx == g_dlen[we]) blk[BLOCK - 3 + q] = ' ';
                else blk[BLOCK - 3 + q] = ' ';
            }
            if (census) census[we]++;
        }
        if (ws >= 0) {
            /* bytes of the straddling plant that lie in this block: word bytes 3.., then ' ' */
            int L = g_dlen[ws];
            for (int q = 3; q < L; q++) blk[q - 3] = (uint8_t)g_dict[ws][q];
            if (L + 1 - 3 > 0) blk[L - 3] = ' ';
        }
    }
    if (pmask) *pmask = mask;
    return 0;
}
