// scan_core.cuh -- the wordcount/grep scan step shared by the sm_100a kernels (gsys_kernels.cu)
// and the host-side emulation used by CPU tests (tests/native/scan_emul.cu).  Part of the CUDA
// path: the oracle (oracle/) never includes it.
//
// Definitions (reading A9/A10): a token is a maximal run of [A-Za-z0-9_]; it is owned
// by the chunk holding its first byte; a dictionary hit is a whole token byte-equal to one of <= 64
// words of <= 16 bytes; grep -F reports whether any pattern occurs as a substring.
#pragma once
#include <cuda_runtime.h>
#include <errno.h>
#include <stdint.h>
#include <string.h>

#ifdef __CUDACC__
#define GSYS_HD __host__ __device__ __forceinline__
#else
#define GSYS_HD inline
#endif

namespace gsys_scan {

#if !defined(__CUDA_ARCH__)
inline int host_ffs(unsigned x) { return x ? __builtin_ctz(x) + 1 : 0; }
inline unsigned host_funnelshift_r(unsigned lo, unsigned hi, unsigned sh) {
    sh &= 31u;
    return sh ? (lo >> sh) | (hi << (32 - sh)) : lo;
}
#define GSYS_FFS host_ffs
#define GSYS_FSHR host_funnelshift_r
#else
#define GSYS_FFS __ffs
#define GSYS_FSHR __funnelshift_r
#endif

constexpr int HBITS = 10;
constexpr int HB = 1 << HBITS;
constexpr int MAXD = 64;
constexpr int MAXP = 8;

struct ScanTables {
    uint4 words[MAXD];          // zero-padded dictionary words
    uint4 pats[MAXP];           // zero-padded grep patterns
    unsigned hmul[5];
    unsigned lenmask;           // bit L: some word has length L
    unsigned ndict, npat;
    unsigned fb_lo, fb_hi;      // first-byte range of patterns (SWAR candidate filter)
    unsigned fbmap[8];          // exact first-byte bitmap
    unsigned char dlen[MAXD];
    unsigned char plen[MAXP];
    unsigned short bucket[HB];  // 0 = empty, else dictionary index + 1
};

// ------------------------------------------------------------------ device helpers
GSYS_HD unsigned compress4(unsigned m80) { return ((m80 >> 7) * 0x10204080u) >> 28; }

// 4-bit mask of bytes of x in [A-Za-z0-9_]
GSYS_HD unsigned class4(unsigned x) {
    unsigned lo7 = x & 0x7f7f7f7fu;
    unsigned y = lo7 | 0x20202020u;                 // ASCII case fold
    unsigned letter = (y + 0x1f1f1f1fu) & ~(y + 0x05050505u);      // 'a'..'z'
    unsigned digit = (lo7 + 0x50505050u) & ~(lo7 + 0x46464646u);   // '0'..'9'
    unsigned t = lo7 ^ 0x5f5f5f5fu;
    unsigned us = ~((t + 0x7f7f7f7fu) | t);                        // '_'
    return compress4((letter | digit | us) & ~x & 0x80808080u);
}
GSYS_HD unsigned class16(uint4 v) {
    return class4(v.x) | (class4(v.y) << 4) | (class4(v.z) << 8) | (class4(v.w) << 12);
}
// 4-bit mask of bytes of x in [lo, hi] (lo <= hi < 0x80)
GSYS_HD unsigned range4(unsigned x, unsigned add_lo, unsigned add_hi) {
    unsigned lo7 = x & 0x7f7f7f7fu;
    return compress4((lo7 + add_lo) & ~(lo7 + add_hi) & ~x & 0x80808080u);
}
GSYS_HD bool is_word_byte(unsigned c) {
    return (c - 'a' < 26u) || (c - 'A' < 26u) || (c - '0' < 10u) || c == '_';
}

// 16 bytes of the 32-byte window (A, B) starting at byte j (0..15), little-endian
GSYS_HD void extract16(const uint4& A, const uint4& B, unsigned j, unsigned t[4]) {
    const bool s8 = j & 8, s4 = j & 4;
    unsigned u0 = s8 ? A.z : A.x, u1 = s8 ? A.w : A.y, u2 = s8 ? B.x : A.z;
    unsigned u3 = s8 ? B.y : A.w, u4 = s8 ? B.z : B.x, u5 = s8 ? B.w : B.y;
    unsigned v0 = s4 ? u1 : u0, v1 = s4 ? u2 : u1, v2 = s4 ? u3 : u2, v3 = s4 ? u4 : u3, v4 = s4 ? u5 : u4;
    unsigned sh = (j & 3u) * 8u;
    t[0] = GSYS_FSHR(v0, v1, sh);
    t[1] = GSYS_FSHR(v1, v2, sh);
    t[2] = GSYS_FSHR(v2, v3, sh);
    t[3] = GSYS_FSHR(v3, v4, sh);
}
GSYS_HD void mask_len(unsigned t[4], unsigned len) {
#pragma unroll
    for (int k = 0; k < 4; k++) {
        int kept = (int)len - 4 * k;
        kept = kept < 0 ? 0 : (kept > 4 ? 4 : kept);
        unsigned m = kept >= 4 ? 0xffffffffu : ((1u << (8 * kept)) - 1u);
        t[k] &= m;
    }
}


// One 16-byte step of the scan at text position p0 (16-byte aligned relative to the chunk):
//   A = bytes [p0, p0+16), B = bytes [p0+16, p0+32) (zeros past valid_end), prevb = byte p0-1
//   (only meaningful when p0 > 0).  Owned token starts are positions in [p0, min(p0+16, own_end));
//   bytes at or beyond valid_end do not exist (end of file / short read).
// on_word(d) is called once per whole-token hit of dictionary word d; the return value is true
// if a grep pattern starts at an owned position (only evaluated when grep is true).
template <class OnWord>
GSYS_HD bool scan_step(const ScanTables& T, const uint4& A, const uint4& B, unsigned prevb, long long p0,
                       long long own_end, long long valid_end, bool grep, OnWord&& on_word) {
    unsigned M = class16(A) | (class16(B) << 16);
    const long long nvalid = valid_end - p0;
    if (nvalid < 32) M &= (1u << nvalid) - 1u;
    const unsigned prevw = (p0 > 0 && is_word_byte(prevb)) ? 1u : 0u;
    const long long nown = own_end - p0;
    const unsigned ownm = nown >= 16 ? 0xffffu : ((1u << nown) - 1u);
    unsigned starts = M & ~((M << 1) | prevw) & ownm;
    while (starts) {
        const unsigned j = GSYS_FFS(starts) - 1u;
        starts &= starts - 1u;
        const unsigned len = (unsigned)GSYS_FFS(~(M >> j)) - 1u;
        if (len > 16u || !((T.lenmask >> len) & 1u)) continue;
        unsigned t[4];
        extract16(A, B, j, t);
        mask_len(t, len);
        const unsigned h = (t[0] * T.hmul[0] + t[1] * T.hmul[1] + t[2] * T.hmul[2] + t[3] * T.hmul[3] +
                            len * T.hmul[4]) >> (32 - HBITS);
        const unsigned b = T.bucket[h];
        if (b) {
            const unsigned d = b - 1u;
            const uint4 w = T.words[d];
            if (T.dlen[d] == len && w.x == t[0] && w.y == t[1] && w.z == t[2] && w.w == t[3]) on_word(d);
        }
    }
    if (!grep) return false;
    const bool fb_swar = T.fb_hi < 0x80u;
    const unsigned add_lo = (0x80u - T.fb_lo) * 0x01010101u, add_hi = (0x7fu - T.fb_hi) * 0x01010101u;
    unsigned cand = fb_swar ? (range4(A.x, add_lo, add_hi) | (range4(A.y, add_lo, add_hi) << 4) |
                               (range4(A.z, add_lo, add_hi) << 8) | (range4(A.w, add_lo, add_hi) << 12))
                            : 0xffffu;
    cand &= ownm;
    while (cand) {
        const unsigned j = GSYS_FFS(cand) - 1u;
        cand &= cand - 1u;
        const unsigned c0 = ((j < 4 ? A.x : j < 8 ? A.y : j < 12 ? A.z : A.w) >> (8 * (j & 3))) & 0xffu;
        if (!((T.fbmap[c0 >> 5] >> (c0 & 31)) & 1u)) continue;
        unsigned t[4];
        extract16(A, B, j, t);
        for (unsigned p = 0; p < T.npat; p++) {
            const unsigned L = T.plen[p];
            if ((long long)(j + L) > nvalid) continue;
            unsigned u[4] = {t[0], t[1], t[2], t[3]};
            mask_len(u, L);
            const uint4 w = T.pats[p];
            if (w.x == u[0] && w.y == u[1] && w.z == u[2] && w.w == u[3]) return true;
        }
    }
    return false;
}

// ------------------------------------------------------------------ host: table builder
inline uint32_t lcg_next(uint64_t* s) {
    *s = *s * 6364136223846793005ull + 1442695040888963407ull;
    return (uint32_t)(*s >> 32);
}

inline unsigned hash_host(const uint32_t t[4], unsigned len, const unsigned m[5]) {
    return (t[0] * m[0] + t[1] * m[1] + t[2] * m[2] + t[3] * m[3] + len * m[4]) >> (32 - HBITS);
}

inline int build_tables(ScanTables* T, const char* dict, const uint8_t* dlen, uint32_t ndict, const char* pats,
                 const uint8_t* plen, uint32_t npat) {
    if (ndict > (uint32_t)MAXD || npat > (uint32_t)MAXP) return -EINVAL;
    if (ndict && (!dict || !dlen)) return -EINVAL;
    if (npat && (!pats || !plen)) return -EINVAL;
    memset(T, 0, sizeof *T);
    T->ndict = ndict;
    T->npat = npat;
    uint32_t w[MAXD][4];
    for (uint32_t d = 0; d < ndict; d++) {
        if (dlen[d] < 1 || dlen[d] > 16) return -EINVAL;
        uint8_t b[16] = {0};
        memcpy(b, dict + 17 * d, dlen[d]);
        memcpy(w[d], b, 16);
        memcpy(&T->words[d], b, 16);
        T->dlen[d] = dlen[d];
        T->lenmask |= 1u << dlen[d];
    }
    uint64_t seed = 0x9E3779B97F4A7C15ull;
    for (int attempt = 0;; attempt++) {
        if (attempt > 100000) return -EINVAL;   // duplicate dictionary words
        for (int k = 0; k < 5; k++) T->hmul[k] = lcg_next(&seed) | 1u;
        memset(T->bucket, 0, sizeof T->bucket);
        bool ok = true;
        for (uint32_t d = 0; d < ndict && ok; d++) {
            unsigned h = hash_host(w[d], dlen[d], T->hmul);
            if (T->bucket[h]) ok = false;
            else T->bucket[h] = (unsigned short)(d + 1);
        }
        if (ok) break;
    }
    T->fb_lo = 0xff;
    T->fb_hi = 0;
    for (uint32_t p = 0; p < npat; p++) {
        if (plen[p] < 1 || plen[p] > 16) return -EINVAL;
        uint8_t b[16] = {0};
        memcpy(b, pats + 17 * p, plen[p]);
        memcpy(&T->pats[p], b, 16);
        T->plen[p] = plen[p];
        unsigned c = b[0];
        T->fbmap[c >> 5] |= 1u << (c & 31);
        if (c < T->fb_lo) T->fb_lo = c;
        if (c > T->fb_hi) T->fb_hi = c;
    }
    if (npat == 0) { T->fb_lo = 0; T->fb_hi = 0; }
    return 0;
}

}  // namespace gsys_scan
