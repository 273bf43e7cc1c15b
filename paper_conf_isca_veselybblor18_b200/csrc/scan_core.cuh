// scan_core.cuh -- the wordcount/grep scan step shared by the sm_100a kernels (gsys_kernels.cu)
// and the host-side emulation used by CPU tests (tests/native/scan_emul.cu).  Part of the CUDA
// path: the oracle (oracle/) never includes it.
//
// Definitions (reading A9/A10): a token is a maximal run of [A-Za-z0-9_]; it is owned
// by the chunk holding its first byte; a dictionary hit is a whole token byte-equal to one of <= 64
// words of <= 16 bytes; grep -F reports whether any pattern occurs as a substring.
//
// Wordcount runs a byte-level DFA built from a trie of the dictionary ("search for occurrences of
// 64 strings", PAPER.md:32 P32.6): state ROOT (at a token start), DEAD (inside a token that can no
// longer match) and one state per dictionary prefix.  A byte b selects column clamp(b-47, 0, 76):
// column 0 holds every byte <= '/', 76 every byte >= '{', 1..75 the bytes '0'..'z' one by one, so
// the table needs 77 columns and no class lookup.  A non-word byte leaves any state for ROOT and,
// from a state that spells a whole dictionary word, emits that word.  Entry (u16) = next state in
// bits 0..8 (<= 512 states) | (word+1) in bits 9..15 (terminating entries only; their next state
// is ROOT = 0), so one shared-memory load, one AND and one shift per byte, no per-token branch.
// Hits are counted with a predicated shared-memory reduction on the device (no divergence).  Two
// segments run interleaved per lane (two independent state chains) to hide the load latency.
// grep keeps a SWAR first-byte range filter plus a 128-bit verify per candidate.
#pragma once
#include <cuda_runtime.h>
#include <errno.h>
#include <stdint.h>
#include <string.h>

#include <vector>

#ifdef __CUDACC__
#define GSYS_HD __host__ __device__ __forceinline__
#else
#define GSYS_HD inline
#endif
#ifdef __CUDA_ARCH__
#define GSYS_UNROLL _Pragma("unroll")
#else
#define GSYS_UNROLL
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

constexpr int MAXD = 64;
constexpr int MAXP = 8;
constexpr int NCOL = 77;                 // DFA columns (see header)
constexpr unsigned ROOT = 0u, DEAD = 1u;
constexpr unsigned MAX_STATES = 512;    // 9-bit next-state field

struct ScanTables {
    uint4 pats[MAXP];           // zero-padded grep patterns
    unsigned ndict, npat;
    unsigned nstates;           // DFA states; the table (nstates x NCOL u16) follows the struct
    unsigned fb_lo, fb_hi;      // first-byte range of patterns (SWAR candidate filter)
    unsigned fbmap[8];          // exact first-byte bitmap
    unsigned char plen[MAXP];
    unsigned pad_[2];
};
static_assert(sizeof(ScanTables) % 16 == 0, "ScanTables must keep the DFA 16-byte aligned");

GSYS_HD size_t tables_bytes(unsigned nstates) { return sizeof(ScanTables) + (size_t)nstates * NCOL * 2; }

// ------------------------------------------------------------------ helpers
GSYS_HD unsigned compress4(unsigned m80) { return ((m80 >> 7) * 0x10204080u) >> 28; }

// 4-bit mask of bytes of x in [lo, hi] (lo <= hi < 0x80)
GSYS_HD unsigned range4(unsigned x, unsigned add_lo, unsigned add_hi) {
    unsigned lo7 = x & 0x7f7f7f7fu;
    return compress4((lo7 + add_lo) & ~(lo7 + add_hi) & ~x & 0x80808080u);
}
GSYS_HD bool is_word_byte(unsigned c) {
    return (c - 'a' < 26u) || (c - 'A' < 26u) || (c - '0' < 10u) || c == '_';
}
GSYS_HD unsigned dfa_col(unsigned b) {
    int c = (int)b - 47;
    c = c < 0 ? 0 : c;
    return (unsigned)(c > NCOL - 1 ? NCOL - 1 : c);
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
    for (int k = 0; k < 4; k++) {
        int kept = (int)len - 4 * k;
        kept = kept < 0 ? 0 : (kept > 4 ? 4 : kept);
        unsigned m = kept >= 4 ? 0xffffffffu : ((1u << (8 * kept)) - 1u);
        t[k] &= m;
    }
}
// byte i (0..31) of the window (A, B)
GSYS_HD unsigned window_byte(const uint4& A, const uint4& B, unsigned i) {
    const unsigned q = i >> 2;
    const unsigned w = q < 4 ? (q < 2 ? (q == 0 ? A.x : A.y) : (q == 2 ? A.z : A.w))
                             : (q < 6 ? (q == 4 ? B.x : B.y) : (q == 6 ? B.z : B.w));
    return (w >> (8 * (i & 3u))) & 0xffu;
}

// One DFA transition; returns the word id + 1 emitted (0 = none).
GSYS_HD unsigned dfa_step(const unsigned short* __restrict__ dfa, unsigned& st, unsigned b) {
    const unsigned e = dfa[st * NCOL + dfa_col(b)];
    st = e & 0x1ffu;
    return e >> 9;
}

// Start state of a step at p0: inside a token owned by the left neighbour -> DEAD.
GSYS_HD unsigned start_state(unsigned prevb, long long p0) {
    return (p0 > 0 && is_word_byte(prevb)) ? DEAD : ROOT;
}

// Follow the token still open after owned byte index `from` of window (A, B) to its end.
template <class OnHit>
GSYS_HD void dfa_finish(const unsigned short* __restrict__ dfa, unsigned st, const uint4& A, const uint4& B,
                        unsigned from, unsigned nvalid, OnHit&& on_hit) {
    for (unsigned i = from; st > DEAD; i++) {
        const unsigned b = i < nvalid ? window_byte(A, B, i) : 0u;   // past the data: terminator
        on_hit(dfa_step(dfa, st, b));
        if (i >= nvalid) break;
    }
}

// Two full 16-byte steps (both owned and valid for all 16 bytes) run interleaved.
template <class OnHit>
GSYS_HD void dfa_pair(const unsigned short* __restrict__ dfa, unsigned& s0, unsigned& s1, const uint4& A0,
                      const uint4& A1, OnHit&& on_hit) {
    const unsigned w0[4] = {A0.x, A0.y, A0.z, A0.w};
    const unsigned w1[4] = {A1.x, A1.y, A1.z, A1.w};
GSYS_UNROLL
    for (int i = 0; i < 16; i++) {
        const unsigned h0 = dfa_step(dfa, s0, (w0[i >> 2] >> (8 * (i & 3))) & 0xffu);
        const unsigned h1 = dfa_step(dfa, s1, (w1[i >> 2] >> (8 * (i & 3))) & 0xffu);
        on_hit(h0);
        on_hit(h1);
    }
}

// One 16-byte step of the scan at text position p0:
//   A = bytes [p0, p0+16), B = bytes [p0+16, p0+32) (zeros past valid_end), prevb = byte p0-1
//   (meaningful when p0 > 0).  Owned token starts are the positions [p0, min(p0+16, own_end));
//   a token owned here is followed into B until it ends (at most 16 + 1 bytes); bytes at or past
//   valid_end do not exist (end of file / short read) and terminate the token.
// on_hit(h) receives every DFA emission value (h = word id + 1, or 0 for none) -- the device
// counts with a predicated reduction, the host emulation with a branch.
template <class OnHit>
GSYS_HD void dfa_segment(const unsigned short* __restrict__ dfa, const uint4& A, const uint4& B, unsigned prevb,
                         long long p0, long long own_end, long long valid_end, OnHit&& on_hit) {
    const long long nvalid_ll = valid_end - p0;
    const unsigned nvalid = nvalid_ll >= 32 ? 32u : (unsigned)nvalid_ll;
    const long long nown_ll = own_end - p0;
    const unsigned nown = nown_ll >= 16 ? 16u : (unsigned)nown_ll;
    unsigned st = start_state(prevb, p0);
    for (unsigned i = 0; i < nown && i < nvalid; i++) on_hit(dfa_step(dfa, st, window_byte(A, B, i)));
    dfa_finish(dfa, st, A, B, nown, nvalid, on_hit);
}

// grep part of a step: true if a pattern starts at an owned position of [p0, p0+16).
GSYS_HD bool grep_step(const ScanTables& T, const uint4& A, const uint4& B, long long p0, long long own_end,
                       long long valid_end) {
    const long long nvalid_ll = valid_end - p0;
    const unsigned nvalid = nvalid_ll >= 32 ? 32u : (unsigned)nvalid_ll;
    const long long nown_ll = own_end - p0;
    const unsigned nown = nown_ll >= 16 ? 16u : (unsigned)nown_ll;
    const bool fb_swar = T.fb_hi < 0x80u;
    const unsigned add_lo = (0x80u - T.fb_lo) * 0x01010101u, add_hi = (0x7fu - T.fb_hi) * 0x01010101u;
    unsigned cand = fb_swar ? (range4(A.x, add_lo, add_hi) | (range4(A.y, add_lo, add_hi) << 4) |
                               (range4(A.z, add_lo, add_hi) << 8) | (range4(A.w, add_lo, add_hi) << 12))
                            : 0xffffu;
    cand &= nown >= 16u ? 0xffffu : ((1u << nown) - 1u);
    while (cand) {
        const unsigned j = GSYS_FFS(cand) - 1u;
        cand &= cand - 1u;
        const unsigned c0 = window_byte(A, B, j);
        if (!((T.fbmap[c0 >> 5] >> (c0 & 31)) & 1u)) continue;
        unsigned t[4];
        extract16(A, B, j, t);
        for (unsigned p = 0; p < T.npat; p++) {
            const unsigned L = T.plen[p];
            if (j + L > nvalid) continue;
            unsigned u[4] = {t[0], t[1], t[2], t[3]};
            mask_len(u, L);
            const uint4 w = T.pats[p];
            if (w.x == u[0] && w.y == u[1] && w.z == u[2] && w.w == u[3]) return true;
        }
    }
    return false;
}

// A lane's 80-byte window as five named vectors (never an indexed array, so it stays in registers)
struct Win {
    uint4 w0, w1, w2, w3, w4;
    GSYS_HD uint4 get(unsigned k) const {   // by value: component-wise selects, no addressable array
        uint4 r = w4;
        if (k == 3) r = w3;
        if (k == 2) r = w2;
        if (k == 1) r = w1;
        if (k == 0) r = w0;
        return r;
    }
};

// byte i (0..79) of the window
GSYS_HD unsigned lane_byte(const Win& W, unsigned i) {
    const uint4 a = W.get(i >> 4);
    return window_byte(a, a, i & 15u);
}

// A lane's 64-byte span at p0: W[0..3] = bytes [p0, p0+64), W[4] = [p0+64, p0+80) (zeros past
// valid_end).  Owned token starts: [p0, min(p0+64, own_end)); the token open at the end of the
// owned range is followed to its end (<= 17 more bytes, all inside W[4] for a full span).
template <class OnHit>
GSYS_HD void dfa_lane64(const unsigned short* __restrict__ dfa, const Win& W, unsigned prevb, long long p0,
                        long long own_end, long long valid_end, OnHit&& on_hit) {
    const long long nvalid_ll = valid_end - p0;
    const unsigned nvalid = nvalid_ll >= 80 ? 80u : (unsigned)nvalid_ll;
    const long long nown_ll = own_end - p0;
    const unsigned nown = nown_ll >= 64 ? 64u : (unsigned)nown_ll;
    unsigned st = start_state(prevb, p0);
    if (nown == 64u && nvalid >= 64u) {
GSYS_UNROLL
        for (int k = 0; k < 4; k++) {
            const uint4 q = W.get((unsigned)k);
            const unsigned wv[4] = {q.x, q.y, q.z, q.w};
GSYS_UNROLL
            for (int i = 0; i < 16; i++) on_hit(dfa_step(dfa, st, (wv[i >> 2] >> (8 * (i & 3))) & 0xffu));
        }
        for (unsigned i = 64; st > DEAD; i++) {
            const unsigned b = i < nvalid ? window_byte(W.w4, W.w4, i - 64u) : 0u;
            on_hit(dfa_step(dfa, st, b));
            if (i >= nvalid) break;
        }
        return;
    }
    for (unsigned i = 0; i < nown && i < nvalid; i++) on_hit(dfa_step(dfa, st, lane_byte(W, i)));
    for (unsigned i = nown; st > DEAD; i++) {
        const unsigned b = i < nvalid ? lane_byte(W, i) : 0u;
        on_hit(dfa_step(dfa, st, b));
        if (i >= nvalid) break;
    }
}

// grep over a lane's span: the four 16-byte steps with their 32-byte windows.
GSYS_HD bool grep_lane64(const ScanTables& T, const Win& W, long long p0, long long own_end, long long valid_end) {
    for (unsigned k = 0; k < 4; k++) {
        const long long q = p0 + 16 * k;
        if (q >= own_end) break;
        const uint4 a = W.get(k), b = W.get(k + 1);
        if (grep_step(T, a, b, q, own_end, valid_end)) return true;
    }
    return false;
}

// Whole step (wordcount + grep) for one segment -- the reference composition used by the host
// emulation; the kernels run the 64-byte lane spans above (checked equal by the CPU tests).
template <class OnHit>
GSYS_HD bool scan_step(const ScanTables& T, const unsigned short* __restrict__ dfa, const uint4& A, const uint4& B,
                       unsigned prevb, long long p0, long long own_end, long long valid_end, bool grep,
                       OnHit&& on_hit) {
    dfa_segment(dfa, A, B, prevb, p0, own_end, valid_end, on_hit);
    return grep && grep_step(T, A, B, p0, own_end, valid_end);
}

// ------------------------------------------------------------------ host: table builder
// Writes ScanTables followed by the DFA (nstates x NCOL u16) into `out` (tables_bytes(nstates)
// bytes, capacity `cap`).  Dictionary words must be 1..16 bytes; a word containing a non-word
// byte can never equal a token and gets no trie path; duplicate words count once (first wins).
// -E2BIG when the trie needs more than 512 states (distinct prefixes + 2).
inline int build_tables(void* out, size_t cap, const char* dict, const uint8_t* dlen, uint32_t ndict,
                        const char* pats, const uint8_t* plen, uint32_t npat, size_t* used) {
    if (ndict > (uint32_t)MAXD || npat > (uint32_t)MAXP) return -EINVAL;
    if (ndict && (!dict || !dlen)) return -EINVAL;
    if (npat && (!pats || !plen)) return -EINVAL;
    // trie over the DFA columns
    std::vector<short> child;            // [state][NCOL]
    std::vector<unsigned char> acc;      // word id + 1 per state
    child.assign(2 * NCOL, -1);
    acc.assign(2, 0);
    for (uint32_t d = 0; d < ndict; d++) {
        if (dlen[d] < 1 || dlen[d] > 16) return -EINVAL;
        const unsigned char* w = (const unsigned char*)dict + 17 * d;
        bool ok = true;
        for (unsigned k = 0; k < dlen[d]; k++) ok = ok && is_word_byte(w[k]);
        if (!ok) continue;
        unsigned s = ROOT;
        for (unsigned k = 0; k < dlen[d]; k++) {
            const unsigned c = dfa_col(w[k]);
            if (child[s * NCOL + c] < 0) {
                child[s * NCOL + c] = (short)acc.size();
                acc.push_back(0);
                child.resize(acc.size() * NCOL, -1);
            }
            s = (unsigned)child[s * NCOL + c];
        }
        if (!acc[s]) acc[s] = (unsigned char)(d + 1);
    }
    const unsigned nstates = (unsigned)acc.size();
    if (nstates > MAX_STATES) return -E2BIG;     // dictionary trie too large for the 9-bit state field
    const size_t need = tables_bytes(nstates);
    if (used) *used = need;
    if (!out || need > cap) return -ENOSPC;
    ScanTables* T = (ScanTables*)out;
    memset(T, 0, sizeof *T);
    T->ndict = ndict;
    T->npat = npat;
    T->nstates = nstates;
    unsigned short* dfa = (unsigned short*)((unsigned char*)out + sizeof(ScanTables));
    for (unsigned s = 0; s < nstates; s++) {
        for (unsigned c = 0; c < (unsigned)NCOL; c++) {
            const unsigned b = c == 0 ? 0u : (c == NCOL - 1 ? 255u : c + 47u);   // a byte of the column
            unsigned short e;
            if (!is_word_byte(b)) e = (unsigned short)((s >= 2 ? acc[s] : 0u) << 9);
            else if (s == DEAD) e = (unsigned short)DEAD;
            else e = child[s * NCOL + c] >= 0 ? (unsigned short)child[s * NCOL + c] : (unsigned short)DEAD;
            dfa[s * NCOL + c] = e;
        }
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
