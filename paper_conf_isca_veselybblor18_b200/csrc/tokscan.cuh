// tokscan.cuh -- token-level wordcount step (row a8, SURVEY.md sec. 8a "SWAR token starts ->
// length filter -> verify against the dictionary"), shared by the sm_100a kernels
// (gsys_kernels.cu) and the host emulation used by CPU tests (tests/native/scan_emul.cu).  Part of
// the CUDA path: the oracle (oracle/) never includes it.
//
// Same definitions as scan_core.cuh (reading A9/A10): a token is a maximal run of [A-Za-z0-9_],
// owned by the chunk holding its first byte; a dictionary hit is a whole token byte-equal to one
// of <= 64 words of <= 16 bytes ("search for occurrences of 64 strings", PAPER.md:32 P32.6).
//
// Instead of one DFA lookup per byte (scan_core.cuh: a shared-memory gather per byte, bound by
// bank conflicts), a lane classifies its 64-byte span four bytes per SWAR step into a 64-bit
// word-byte mask, derives the token starts with two shifts, and visits only the tokens: the
// length comes from the mask (one count-trailing-zeros), tokens of a length no dictionary word
// has are skipped, the first 8 (16) bytes are read from the staged span, hashed, and looked up in a
// collision-free hash table of the dictionary (the builder picks multipliers until the words land
// in distinct slots), then verified byte-exactly -- about four shared-memory accesses per token
// (mean token 5.8 bytes plus separators) instead of one per byte.
#pragma once
#include <stddef.h>

#include "scan_core.cuh"

namespace gsys_tok {

using gsys_scan::Win;
#if !defined(__CUDA_ARCH__)
using gsys_scan::host_funnelshift_r;
#endif
constexpr unsigned HBITS = 10;
constexpr unsigned HSIZE = 1u << HBITS;
constexpr unsigned MAXD = 64;

struct TokTables {
    gsys_scan::ScanTables g;    // grep part (patterns, first-byte filter); its DFA fields are unused
    uint4 key[MAXD];            // word d's bytes 0..15, zero-padded
    unsigned ndict;
    unsigned lenmask;           // bit L: some matchable dictionary word has length L (1..16)
    unsigned m[5];              // hash multipliers (bytes 0-3, 4-7, 8-11, 12-15, length)
    unsigned one;               // 1 (a run-time constant: see word4)
    unsigned char klen[MAXD];
    unsigned char slot[HSIZE];  // 0: empty, else word index + 1
};
static_assert(sizeof(TokTables) % 16 == 0, "TokTables must keep 16-byte alignment");

// Slot of a token: its first 8 bytes (zero-padded) and its length.  The builder requires the
// matchable words to differ in (first 8 bytes, length) -- bytes 8..15 are only verified.
GSYS_HD unsigned tok_hash(const unsigned m[5], unsigned a, unsigned b, unsigned len) {
    return ((a * m[0]) ^ (b * m[1]) ^ (len * m[4])) >> (32u - HBITS);
}

// Word bytes of a little-endian 4-byte group: bit 7 of byte i set iff byte i is in [0-9A-Za-z_]
// (bytes >= 0x80 are not).  Per byte, 7-bit adds that cannot carry across bytes.
// `one` == 1 at run time: the adds become IMADs (x * one + c) and run on the FMA pipe, next to the
// LOP3s on the ALU pipe (the token scan is ALU-pipe bound: B200 issues 16 ALU lanes per SMSP).
GSYS_HD unsigned word4(unsigned w, unsigned one = 1u) {
    const unsigned a = w & 0x7f7f7f7fu;
    const unsigned x = a | 0x20202020u;                  // letters folded to lower case
    const unsigned g1 = x * one + 0x1f1f1f1fu;           // x >= 0x61
    const unsigned g2 = x * one + 0x05050505u;           // x >= 0x7b
    const unsigned g3 = a * one + 0x50505050u;           // a >= 0x30
    const unsigned g4 = a * one + 0x46464646u;           // a >= 0x3a
    const unsigned nu = (a ^ 0x5f5f5f5fu) * one + 0x7f7f7f7fu; // a != '_'
    // letter: x in [0x61, 0x7a] (no digit or '_' maps there); digit: a in [0x30, 0x39]
    const unsigned v = (g1 & ~g2) | (g3 & ~g4);
    return (v | ~nu) & ~w & 0x80808080u;
}

// Four word4() results -> 16-bit mask (bit i = byte i).
GSYS_HD unsigned pack16(unsigned c0, unsigned c1, unsigned c2, unsigned c3) {
#ifdef __CUDA_ARCH__
    // bytes are 0x80 or 0: a byte dot product with weights 1,2,4,8 (16,..,128) gathers 4 (8) bits x 128
    const unsigned lo = __dp4a(c1, 0x80402010u, __dp4a(c0, 0x08040201u, 0u));
    const unsigned hi = __dp4a(c3, 0x80402010u, __dp4a(c2, 0x08040201u, 0u));
    return (lo | (hi << 8)) >> 7;
#else
    unsigned r = 0;
    const unsigned c[4] = {c0, c1, c2, c3};
    for (int k = 0; k < 4; k++)
        for (int i = 0; i < 4; i++) r |= ((c[k] >> (8 * i + 7)) & 1u) << (4 * k + i);
    return r;
#endif
}

GSYS_HD unsigned mask16(const uint4& q, unsigned one = 1u) {
    return pack16(word4(q.x, one), word4(q.y, one), word4(q.z, one), word4(q.w, one));
}

// Word-byte mask of the lane's 64-byte span W.w0..w3 (bit i = byte p0 + i).
GSYS_HD unsigned long long mask64(const Win& W, unsigned one = 1u) {
    const unsigned a = mask16(W.w0, one) | (mask16(W.w1, one) << 16);
    const unsigned b = mask16(W.w2, one) | (mask16(W.w3, one) << 16);
    return (unsigned long long)a | ((unsigned long long)b << 32);
}

GSYS_HD unsigned ctz32(unsigned x) {
#ifdef __CUDA_ARCH__
    return (unsigned)__ffs((int)x) - 1u;
#else
    return (unsigned)__builtin_ctz(x);
#endif
}

GSYS_HD unsigned ctz64(unsigned long long x) {
#ifdef __CUDA_ARCH__
    return (unsigned)__ffsll((long long)x) - 1u;
#else
    return (unsigned)__builtin_ctzll(x);
#endif
}

// The 8 bytes at p (any alignment) as two little-endian u32: two aligned 8-byte loads + funnel
// shifts.  On the device p is a shared-memory address (explicit ld.shared: no generic-address
// resolution per load).
GSYS_HD void load8(const unsigned char* p, unsigned& lo, unsigned& hi) {
#ifdef __CUDA_ARCH__
    const unsigned a = (unsigned)__cvta_generic_to_shared(p);
    const unsigned q = a & ~7u;
    unsigned w0, w1, w2, w3;
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(w0), "=r"(w1) : "r"(q));
    asm volatile("ld.shared.v2.u32 {%0, %1}, [%2+8];" : "=r"(w2), "=r"(w3) : "r"(q));
    const unsigned o = a & 7u;
#else
    const uintptr_t a = (uintptr_t)p;
    const unsigned* qq = reinterpret_cast<const unsigned*>(a & ~(uintptr_t)7);
    const unsigned o = (unsigned)(a & 7u);
    const unsigned w0 = qq[0], w1 = qq[1], w2 = qq[2], w3 = qq[3];
#endif
    const bool s4 = o & 4u;
    const unsigned u0 = s4 ? w1 : w0, u1 = s4 ? w2 : w1, u2 = s4 ? w3 : w2;
    const unsigned sh = (o & 3u) * 8u;
    lo = GSYS_FSHR(u0, u1, sh);
    hi = GSYS_FSHR(u1, u2, sh);
}

// 0xffffffff >> s with s clamped to [0, 32] (32 or more: 0)
GSYS_HD unsigned shr_ones(int s) {
    s = s < 0 ? 0 : s;
#ifdef __CUDA_ARCH__
    unsigned r;
    asm("shr.b32 %0, %1, %2;" : "=r"(r) : "r"(0xffffffffu), "r"((unsigned)s));   // PTX clamps shifts >= 32
    return r;
#else
    return s >= 32 ? 0u : 0xffffffffu >> s;
#endif
}

// Keep the first n (n >= 1) bytes of (lo, hi): bytes 0..3 in lo, 4..7 in hi.
GSYS_HD void keep8(unsigned& lo, unsigned& hi, unsigned n) {
    lo &= shr_ones(32 - 8 * (int)n);
    hi &= shr_ones(64 - 8 * (int)n);
}

// The tokens owned by one lane span.  span: the span's bytes p0.. in memory (at least 96 readable
// bytes; bytes at or past valid_end are never part of a token because the masks exclude them);
// M: word-byte mask of the 64 span bytes; la: the mask of the 16 bytes after them; prev_word:
// byte p0-1 exists and is a word byte.  Owned token starts are [p0, min(p0+64, own_end)); a token
// may run up to 16 bytes into the lookahead (longer ones cannot match).  emit(d): one hit of word d.
// Table fields a lane keeps in registers for the whole scan.
struct TokRegs {
    unsigned lenmask, m0, m1, m4;
    unsigned tabs;   // device: shared-space address of the TokTables (explicit ld.shared lookups)
};
GSYS_HD TokRegs tok_regs(const TokTables& T) {
#ifdef __CUDA_ARCH__
    const unsigned tabs = (unsigned)__cvta_generic_to_shared(&T);
#else
    const unsigned tabs = 0u;
#endif
    return TokRegs{T.lenmask & 0x1fffeu, T.m[0], T.m[1], T.m[4], tabs};
}

// Table lookups: shared-space loads on the device (the generic form recomputes the shared window
// base per access), plain reads on the host.
GSYS_HD unsigned tok_slot(const TokTables& T, const TokRegs& R, unsigned h) {
#ifdef __CUDA_ARCH__
    unsigned v;
    asm("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(R.tabs + (unsigned)offsetof(TokTables, slot) + h));
    return v & 0xffu;
#else
    (void)R;
    return T.slot[h];
#endif
}
GSYS_HD void tok_key(const TokTables& T, const TokRegs& R, unsigned d, uint4& k, unsigned& klen) {
#ifdef __CUDA_ARCH__
    asm("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(k.x), "=r"(k.y), "=r"(k.z), "=r"(k.w)
        : "r"(R.tabs + (unsigned)offsetof(TokTables, key) + 16u * d));
    asm("ld.shared.u8 %0, [%1];" : "=r"(klen) : "r"(R.tabs + (unsigned)offsetof(TokTables, klen) + d));
    klen &= 0xffu;
#else
    (void)R;
    k = T.key[d];
    klen = T.klen[d];
#endif
}

// The tokens starting at the positions set in S (bit q = byte 32*half + q of the span): lo, hi are
// the word-byte mask of that half and of the 32 bytes after it, so the run of word bytes from q is
// one funnel shift away; a token of 32+ word bytes leaves no zero in the window (length > 16).
template <class Emit>
GSYS_HD void tok_visit(const TokTables& T, const TokRegs& R, const unsigned char* span, unsigned half, unsigned S,
                       unsigned lo, unsigned hi, Emit&& emit) {
    while (S) {
        const unsigned q = ctz32(S);
        S &= S - 1u;
        const unsigned w = GSYS_FSHR(lo, hi, q);
        const unsigned len = ~w ? ctz32(~w) : 32u;
        if (!((R.lenmask >> (len & 31u)) & 1u) || len > 16u) continue;
        const unsigned char* t = span + 32u * half + q;
        unsigned a, b;
        load8(t, a, b);
        keep8(a, b, len);
        const unsigned id = tok_slot(T, R, ((a * R.m0) ^ (b * R.m1) ^ (len * R.m4)) >> (32u - HBITS));
        if (!id) continue;
        uint4 k;
        unsigned klen;
        tok_key(T, R, id - 1u, k, klen);
        if (klen != len || k.x != a || k.y != b) continue;
        if (len > 8u) {   // bytes 8..15: only for the few long words
            unsigned c, d;
            load8(t + 8u, c, d);
            keep8(c, d, len - 8u);
            if (k.z != c || k.w != d) continue;
        }
        emit(id - 1u);
    }
}

// The tokens owned by one lane span.  span: the span's bytes p0.. in memory (at least 80 readable
// bytes; bytes at or past valid_end are never part of a token because the masks exclude them);
// M: word-byte mask of the 64 span bytes; la: the mask of the 16 bytes after them; prev_word:
// byte p0-1 exists and is a word byte.  Owned token starts are [p0, min(p0+64, own_end)); a token
// may run up to 16 bytes into the lookahead (longer ones cannot match).  emit(d): one hit of word d.
template <class Emit>
GSYS_HD void tok_lane64(const TokTables& T, const TokRegs& R, const unsigned char* span, unsigned long long M,
                        unsigned la, bool prev_word, long long p0, long long own_end, long long valid_end,
                        Emit&& emit) {
    const long long nvalid_ll = valid_end - p0;
    if (nvalid_ll < 80) {   // end of data: bytes at or past valid_end terminate tokens
        const unsigned nv = nvalid_ll <= 0 ? 0u : (unsigned)nvalid_ll;
        if (nv < 64u) { M &= nv ? (~0ull >> (64u - nv)) : 0ull; la = 0u; }
        else la &= (1u << (nv - 64u)) - 1u;
    }
    const unsigned m0 = (unsigned)M, m1 = (unsigned)(M >> 32), m2 = la & 0xffffu;
    unsigned s0 = m0 & ~((m0 << 1) | (prev_word ? 1u : 0u));
    unsigned s1 = m1 & ~((m1 << 1) | (m0 >> 31));
    const long long nown_ll = own_end - p0;
    if (nown_ll < 64) {
        const unsigned no = nown_ll <= 0 ? 0u : (unsigned)nown_ll;
        s0 &= no >= 32u ? 0xffffffffu : ((1u << no) - 1u);
        s1 &= no <= 32u ? 0u : ((1u << (no - 32u)) - 1u);
    }
    tok_visit(T, R, span, 0u, s0, m0, m1, emit);
    tok_visit(T, R, span, 1u, s1, m1, m2, emit);
}

// ------------------------------------------------------------------ host: table builder
// Dictionary words must be 1..16 bytes; a word containing a non-word byte can never equal a token
// and gets no slot; a duplicate word counts once (the first wins) -- as gsys_scan::build_tables.
// The multipliers are searched (fixed seed) until every matchable word has its own slot.
inline int build_tok_tables(void* out, size_t cap, const char* dict, const uint8_t* dlen, uint32_t ndict,
                            const char* pats, const uint8_t* plen, uint32_t npat, size_t* used) {
    if (ndict > MAXD || npat > (uint32_t)gsys_scan::MAXP) return -EINVAL;
    if (ndict && (!dict || !dlen)) return -EINVAL;
    if (npat && (!pats || !plen)) return -EINVAL;
    if (used) *used = sizeof(TokTables);
    if (!out || cap < sizeof(TokTables)) return -ENOSPC;
    TokTables* T = (TokTables*)out;
    memset(T, 0, sizeof *T);
    T->ndict = ndict;
    T->one = 1u;
    bool match[MAXD] = {false};
    for (uint32_t d = 0; d < ndict; d++) {
        if (dlen[d] < 1 || dlen[d] > 16) return -EINVAL;
        const unsigned char* w = (const unsigned char*)dict + 17 * d;
        uint8_t b[16] = {0};
        memcpy(b, w, dlen[d]);
        memcpy(&T->key[d], b, 16);
        T->klen[d] = dlen[d];
        bool ok = true;
        for (unsigned k = 0; k < dlen[d]; k++) ok = ok && gsys_scan::is_word_byte(w[k]);
        for (uint32_t e = 0; ok && e < d; e++)   // duplicate of an earlier word: the first wins
            if (match[e] && T->klen[e] == dlen[d] && memcmp(&T->key[e], &T->key[d], 16) == 0) ok = false;
        match[d] = ok;
        if (ok) T->lenmask |= 1u << dlen[d];
    }
    // the slot is chosen by (first 8 bytes, length): two matchable words sharing both cannot be told
    // apart by the table -- the byte DFA handles such dictionaries
    for (uint32_t d = 0; d < ndict; d++)
        for (uint32_t e = 0; match[d] && e < d; e++)
            if (match[e] && T->klen[e] == T->klen[d] && T->key[e].x == T->key[d].x && T->key[e].y == T->key[d].y)
                return -E2BIG;
    unsigned long long x = 0x9E3779B97F4A7C15ull;
    bool placed = false;
    for (int attempt = 0; attempt < 100000 && !placed; attempt++) {
        for (int i = 0; i < 5; i++) {
            x ^= x << 13; x ^= x >> 7; x ^= x << 17;
            T->m[i] = (unsigned)(x >> 17) | 1u;
        }
        memset(T->slot, 0, sizeof T->slot);
        placed = true;
        for (uint32_t d = 0; d < ndict && placed; d++) {
            if (!match[d]) continue;
            const uint4 k = T->key[d];
            const unsigned h = tok_hash(T->m, k.x, k.y, T->klen[d]);
            if (T->slot[h]) placed = false;
            else T->slot[h] = (unsigned char)(d + 1);
        }
    }
    if (!placed) return -E2BIG;
    // grep part (same fields and filter as gsys_scan::build_tables)
    gsys_scan::ScanTables& G = T->g;
    G.ndict = ndict;
    G.npat = npat;
    G.fb_lo = 0xff;
    G.fb_hi = 0;
    for (uint32_t p = 0; p < npat; p++) {
        if (plen[p] < 1 || plen[p] > 16) return -EINVAL;
        uint8_t b[16] = {0};
        memcpy(b, pats + 17 * p, plen[p]);
        memcpy(&G.pats[p], b, 16);
        G.plen[p] = plen[p];
        const unsigned c = b[0];
        G.fbmap[c >> 5] |= 1u << (c & 31);
        if (c < G.fb_lo) G.fb_lo = c;
        if (c > G.fb_hi) G.fb_hi = c;
    }
    if (npat == 0) { G.fb_lo = 0; G.fb_hi = 0; }
    return 0;
}

}  // namespace gsys_tok
