// scan_core.cuh -- the wordcount/grep scan step shared by the sm_100a kernels (gsys_kernels.cu)
// and the host-side emulation used by CPU tests (tests/native/scan_emul.cu).  Part of the CUDA
// path: the oracle (oracle/) never includes it.
//
// Definitions (reading A9/A10): a token is a maximal run of [A-Za-z0-9_]; it is owned
// by the chunk holding its first byte; a dictionary hit is a whole token byte-equal to one of <= 64
// words of <= 16 bytes; grep -F reports whether any pattern occurs as a substring.
//
// Wordcount runs a byte-level DFA built from a trie of the dictionary ("search for occurrences of
// 64 strings", PAPER.md:32 P32.6).  States: ROOT (at a token start), DEAD (inside a token that can
// no longer match), one state per dictionary prefix, and one EMISSION state per dictionary word --
// a copy of ROOT entered on the non-word byte that ends a token spelling that word.  Counting a
// hit is therefore "the DFA entered emission state E_d", with no separate output field.
//
// Table layout (transposed, column-major): entry(col, state) is a u16 at byte offset
// col * (2 * nsp) + 2 * state, and the entry's value is 2 * next_state -- the byte offset of the
// next state inside any column.  One transition is one IMAD (col * stride + entry) and one LDS.U16.
// nsp (states per column, padded) is = 2 mod 4, so the column stride is an odd number of 32-bit
// words and lanes sitting in the same state but reading different bytes land on different banks.
// Emission states are numbered last, so "entry >= emit2" (= 2 * first emission state) detects a
// hit and, since two emissions are never adjacent (a token has >= 1 byte), the larger entry of a
// byte pair carries the pair's only possible emission: one compare + one predicated shared RED per
// two bytes.  Two column maps:
//   narrow (77 columns): column = clamp(b - 47, 0, 76) -- bytes <= '/' share column 0, bytes >= '{'
//     column 76 (fits 2 work-groups per SM next to the wordcount's staging);
//   wide (129 columns): column = b for b < 0x80, 128 for any byte >= 0x80; a 64-byte span without
//     a high byte (the common case, checked with one OR tree) indexes the table with the raw byte.
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
constexpr unsigned NCOL_NARROW = 77;    // see header
constexpr unsigned NCOL_WIDE = 129;
constexpr unsigned ROOT = 0u, DEAD = 1u;
constexpr unsigned MAX_TRIE = 512;      // trie states (ROOT, DEAD, dictionary prefixes)

struct ScanTables {
    uint4 pats[MAXP];           // zero-padded grep patterns
    unsigned ndict, npat;
    unsigned nstates;           // trie states; emission state of word d is nstates + d
    unsigned ncol;              // NCOL_NARROW or NCOL_WIDE
    unsigned nsp;               // states per column incl. padding (= 2 mod 4)
    unsigned emit2;             // 2 * nstates: entries >= emit2 are emissions
    unsigned fb_lo, fb_hi;      // first-byte range of patterns (SWAR candidate filter)
    unsigned fbmap[8];          // exact first-byte bitmap
    unsigned char plen[MAXP];
    unsigned pad_[2];
};
static_assert(sizeof(ScanTables) % 16 == 0, "ScanTables must keep the DFA 16-byte aligned");

GSYS_HD size_t tables_bytes(unsigned nsp, unsigned ncol) { return sizeof(ScanTables) + (size_t)ncol * nsp * 2; }

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
GSYS_HD unsigned col_narrow(unsigned b) {
    int c = (int)b - 47;
    c = c < 0 ? 0 : c;
    return (unsigned)(c > (int)NCOL_NARROW - 1 ? (int)NCOL_NARROW - 1 : c);
}
GSYS_HD unsigned col_wide(unsigned b) { return b < 128u ? b : 128u; }

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
// byte i (0..3) of w, zero-extended (one PRMT on the device)
GSYS_HD unsigned byte_of(unsigned w, unsigned i) {
#ifdef __CUDA_ARCH__
    return __byte_perm(w, 0u, 0x4440u + i);
#else
    return (w >> (8u * i)) & 0xffu;
#endif
}
// warp-uniform "does any active lane still need this" (a lane's own flag on the host)
GSYS_HD bool any_lane(bool p) {
#ifdef __CUDA_ARCH__
    return __any_sync(__activemask(), p);
#else
    return p;
#endif
}
// byte i (0..31) of the window (A, B)
GSYS_HD unsigned window_byte(const uint4& A, const uint4& B, unsigned i) {
    const unsigned q = i >> 2;
    const unsigned w = q < 4 ? (q < 2 ? (q == 0 ? A.x : A.y) : (q == 2 ? A.z : A.w))
                             : (q < 6 ? (q == 4 ? B.x : B.y) : (q == 6 ? B.z : B.w));
    return (w >> (8 * (i & 3u))) & 0xffu;
}

// View of the transposed DFA (see header).  Entries are org + 2 * state; the DFA "state" carried
// by the scan is the entry value itself.  Host (emulation): org = 0 and entry(col, e) is read at
// base + col * stride + e.  Device: the kernel adds org = the shared-window address of column 0 to
// every entry when it stages the table (load_tables), so col * stride + e IS the shared address of
// the next entry -- one IMAD and one LDS.U16 per byte, no base add.
template <bool WIDE>
struct Dfa {
    const unsigned char* base;  // host: entry(col, e) at base + col * stride + e
    unsigned stride;            // 2 * nsp
    unsigned emit2;             // first emission entry (org + 2 * nstates)
    unsigned org;               // entry of state 0 (ROOT)
    GSYS_HD static unsigned col(unsigned b) { return WIDE ? col_wide(b) : col_narrow(b); }
    GSYS_HD unsigned at(unsigned c, unsigned e) const {
#ifdef __CUDA_ARCH__
        unsigned v;
        asm volatile("ld.shared.u16 %0, [%1];" : "=r"(v) : "r"(c * stride + e));
        return v;
#else
        return *reinterpret_cast<const unsigned short*>(base + c * stride + e);
#endif
    }
    GSYS_HD unsigned step(unsigned e, unsigned b) const { return at(col(b), e); }
    GSYS_HD unsigned root() const { return org + 2u * ROOT; }
    GSYS_HD unsigned dead() const { return org + 2u * DEAD; }
    // inside a token whose prefix is still a dictionary prefix (ROOT, DEAD, emissions are not)
    GSYS_HD bool live(unsigned e) const { return e > dead() && e < emit2; }
};
// Host view (org = 0) of a table in memory.
template <bool WIDE>
GSYS_HD Dfa<WIDE> dfa_view(const ScanTables& T) {
    return Dfa<WIDE>{reinterpret_cast<const unsigned char*>(&T) + sizeof(ScanTables), 2u * T.nsp, T.emit2, 0u};
}
#ifdef __CUDACC__
// Device view of a table staged in shared memory whose entries were rebased by org (see Dfa).
template <bool WIDE>
__device__ __forceinline__ Dfa<WIDE> dfa_view_shared(const ScanTables& T) {
    const unsigned org = (unsigned)__cvta_generic_to_shared(&T) + (unsigned)sizeof(ScanTables);
    return Dfa<WIDE>{nullptr, 2u * T.nsp, org + T.emit2, org};
}
#endif

// Start entry of a span at p0: inside a token owned by the left neighbour -> DEAD.
template <bool WIDE>
GSYS_HD unsigned start_entry(const Dfa<WIDE>& D, unsigned prevb, long long p0) {
    return (p0 > 0 && is_word_byte(prevb)) ? D.dead() : D.root();
}

// One 16-byte step of the scan at text position p0 (the reference composition, host emulation):
//   A = bytes [p0, p0+16), B = bytes [p0+16, p0+32) (zeros past valid_end), prevb = byte p0-1
//   (meaningful when p0 > 0).  Owned token starts are the positions [p0, min(p0+16, own_end));
//   a token owned here is followed into B until it ends (at most 16 more bytes); bytes at or past
//   valid_end do not exist (end of file / short read) and terminate the token.
// emit(e) receives DFA entries; entries >= emit2 are hits of word (e - emit2) / 2.
template <bool WIDE, class Emit>
GSYS_HD void dfa_segment(const Dfa<WIDE>& D, const uint4& A, const uint4& B, unsigned prevb, long long p0,
                         long long own_end, long long valid_end, Emit&& emit) {
    const long long nvalid_ll = valid_end - p0;
    const unsigned nvalid = nvalid_ll >= 32 ? 32u : (unsigned)nvalid_ll;
    const long long nown_ll = own_end - p0;
    const unsigned nown = nown_ll >= 16 ? 16u : (unsigned)nown_ll;
    unsigned e = start_entry(D, prevb, p0);
    for (unsigned i = 0; i < nown && i < nvalid; i++) {
        e = D.step(e, window_byte(A, B, i));
        emit(e);
    }
    for (unsigned i = nown; D.live(e) && i < 32u; i++) {
        const unsigned b = i < nvalid ? window_byte(A, B, i) : 0u;   // past the data: terminator
        e = D.step(e, b);
        emit(e);
        if (i >= nvalid) break;
    }
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

// Transitions over the 64 bytes of W.w0..w3 (all owned and valid), emissions counted per 4 bytes.  RAW: every
// byte is < 0x80 and the table is wide, so the byte is its own column.
// emit2x(hi, lo): count hi if it is an emission, then lo (lo <= hi, rarely an emission).
template <bool RAW, bool WIDE, class Emit2>
GSYS_HD unsigned dfa_run64(const Dfa<WIDE>& D, const Win& W, unsigned e, Emit2&& emit2x) {
GSYS_UNROLL
    for (int k = 0; k < 4; k++) {
        const uint4 q = W.get((unsigned)k);
        const unsigned wv[4] = {q.x, q.y, q.z, q.w};
GSYS_UNROLL
        for (int j = 0; j < 4; j++) {
            const unsigned w = wv[j];
            const unsigned b0 = byte_of(w, 0u), b1 = byte_of(w, 1u), b2 = byte_of(w, 2u), b3 = byte_of(w, 3u);
            const unsigned e0 = D.at(RAW ? b0 : D.col(b0), e);
            const unsigned e1 = D.at(RAW ? b1 : D.col(b1), e0);
            const unsigned e2 = D.at(RAW ? b2 : D.col(b2), e1);
            e = D.at(RAW ? b3 : D.col(b3), e2);
            // at most one of two consecutive entries is an emission, so each pair's larger entry
            // carries its pair's emission; both pairs emit only around a 1-2 byte token
            const unsigned m01 = e0 > e1 ? e0 : e1, m23 = e2 > e ? e2 : e;
            emit2x(m01 > m23 ? m01 : m23, m01 > m23 ? m23 : m01);
        }
    }
    return e;
}

// A lane's 64-byte span at p0: W[0..3] = bytes [p0, p0+64), W[4] = [p0+64, p0+80) (zeros past
// valid_end).  Owned token starts: [p0, min(p0+64, own_end)); the token open at the end of the
// owned range is followed to its end (a live prefix has <= 16 bytes, so it is resolved within the
// 16 bytes of W[4]; a byte at or past valid_end is a terminator).
template <bool WIDE, class Emit, class Emit2>
GSYS_HD void dfa_lane64(const Dfa<WIDE>& D, const Win& W, unsigned prevb, long long p0, long long own_end,
                        long long valid_end, Emit&& emit, Emit2&& emit2x) {
    const long long nvalid_ll = valid_end - p0;
    const unsigned nvalid = nvalid_ll >= 80 ? 80u : (unsigned)nvalid_ll;
    const long long nown_ll = own_end - p0;
    const unsigned nown = nown_ll >= 64 ? 64u : (unsigned)nown_ll;
    unsigned e = start_entry(D, prevb, p0);
    if (nown == 64u && nvalid >= 64u) {
        bool raw = false;
        if (WIDE) {
            const unsigned o = W.w0.x | W.w0.y | W.w0.z | W.w0.w | W.w1.x | W.w1.y | W.w1.z | W.w1.w | W.w2.x |
                               W.w2.y | W.w2.z | W.w2.w | W.w3.x | W.w3.y | W.w3.z | W.w3.w;
            raw = (o & 0x80808080u) == 0u;
        }
        if (raw) e = dfa_run64<true>(D, W, e, emit2x);
        else e = dfa_run64<false>(D, W, e, emit2x);
        if (nvalid == 80u) {
            // follow the open token through W[4] with the entry frozen at its first non-live value
            // (ROOT, DEAD or the word's emission state), then count that one value; a span whose
            // last entry is not live has nothing open (an emission there was counted in the loop)
            const bool lv0 = D.live(e);
            bool lv = lv0;
            const unsigned w4[4] = {W.w4.x, W.w4.y, W.w4.z, W.w4.w};
GSYS_UNROLL
            for (int j = 0; j < 4; j++) {
                if (!any_lane(lv)) break;
GSYS_UNROLL
                for (int i = 0; i < 4; i++) {
                    const unsigned en = D.step(e, byte_of(w4[j], (unsigned)i));
                    e = lv ? en : e;
                    lv = D.live(e);
                }
            }
            emit(lv0 ? e : D.root());
            return;
        }
        const unsigned nla = nvalid - 64u;
        for (unsigned i = 0; i < 16u && D.live(e); i++) {
            const unsigned b = i < nla ? window_byte(W.w4, W.w4, i) : 0u;
            e = D.step(e, b);
            emit(e);
        }
        return;
    }
    for (unsigned i = 0; i < nown && i < nvalid; i++) {
        e = D.step(e, lane_byte(W, i));
        emit(e);
    }
    for (unsigned i = nown; D.live(e) && i <= 80u; i++) {
        const unsigned b = i < nvalid && i < 80u ? lane_byte(W, i) : 0u;
        e = D.step(e, b);
        emit(e);
        if (i >= nvalid) break;
    }
}

// grep's exact part over a lane's span: the four 16-byte steps with their 32-byte windows.
GSYS_HD bool grep_lane64_steps(const ScanTables& T, const Win& W, long long p0, long long own_end,
                               long long valid_end) {
GSYS_UNROLL
    for (int k = 0; k < 4; k++) {
        const long long q = p0 + 16 * k;
        if (q >= own_end) break;
        if (grep_step(T, W.get((unsigned)k), W.get((unsigned)k + 1u), q, own_end, valid_end)) return true;
    }
    return false;
}

// grep over a lane's span: a SWAR first-byte prefilter, then the exact steps.
GSYS_HD bool grep_lane64(const ScanTables& T, const Win& W, long long p0, long long own_end, long long valid_end) {
    if (T.npat == 0) return false;
    if (T.fb_hi < 0x80u) {
        // one SWAR pass over the 64 bytes: does any byte fall in the patterns' first-byte range?
        // (7-bit test: bytes >= 0x80 may pass, the exact steps below reject them)
        const unsigned add_lo = (0x80u - T.fb_lo) * 0x01010101u, add_hi = (0x7fu - T.fb_hi) * 0x01010101u;
        auto r = [add_lo, add_hi](unsigned x) {
            const unsigned lo7 = x & 0x7f7f7f7fu;
            return (lo7 + add_lo) & ~(lo7 + add_hi);
        };
        const unsigned acc = r(W.w0.x) | r(W.w0.y) | r(W.w0.z) | r(W.w0.w) | r(W.w1.x) | r(W.w1.y) | r(W.w1.z) |
                             r(W.w1.w) | r(W.w2.x) | r(W.w2.y) | r(W.w2.z) | r(W.w2.w) | r(W.w3.x) | r(W.w3.y) |
                             r(W.w3.z) | r(W.w3.w);
        if (!(acc & 0x80808080u)) return false;
    }
    return grep_lane64_steps(T, W, p0, own_end, valid_end);
}

// Whole step (wordcount + grep) for one segment -- the reference composition used by the host
// emulation; the kernels run the 64-byte lane spans above (checked equal by the CPU tests).
template <bool WIDE, class Emit>
GSYS_HD bool scan_step(const ScanTables& T, const Dfa<WIDE>& D, const uint4& A, const uint4& B, unsigned prevb,
                       long long p0, long long own_end, long long valid_end, bool grep, Emit&& emit) {
    dfa_segment(D, A, B, prevb, p0, own_end, valid_end, emit);
    return grep && grep_step(T, A, B, p0, own_end, valid_end);
}

// ------------------------------------------------------------------ host: table builder
// Writes ScanTables followed by the transposed DFA (ncol x nsp u16) into `out` (capacity `cap`;
// the size needed is returned in *used).  Dictionary words must be 1..16 bytes; a word containing
// a non-word byte can never equal a token and gets no trie path; duplicate words count once (the
// first wins).  -E2BIG when the trie needs more than MAX_TRIE states (distinct prefixes + 2).
inline int build_tables(void* out, size_t cap, const char* dict, const uint8_t* dlen, uint32_t ndict,
                        const char* pats, const uint8_t* plen, uint32_t npat, size_t* used,
                        unsigned ncol = NCOL_NARROW) {
    if (ndict > (uint32_t)MAXD || npat > (uint32_t)MAXP) return -EINVAL;
    if (ndict && (!dict || !dlen)) return -EINVAL;
    if (npat && (!pats || !plen)) return -EINVAL;
    if (ncol != NCOL_NARROW && ncol != NCOL_WIDE) return -EINVAL;
    // trie over byte values
    std::vector<int> child(2 * 256, -1);   // [state][byte]
    std::vector<unsigned char> acc(2, 0);  // word id + 1 per state
    for (uint32_t d = 0; d < ndict; d++) {
        if (dlen[d] < 1 || dlen[d] > 16) return -EINVAL;
        const unsigned char* w = (const unsigned char*)dict + 17 * d;
        bool ok = true;
        for (unsigned k = 0; k < dlen[d]; k++) ok = ok && is_word_byte(w[k]);
        if (!ok) continue;
        unsigned s = ROOT;
        for (unsigned k = 0; k < dlen[d]; k++) {
            if (child[s * 256 + w[k]] < 0) {
                child[s * 256 + w[k]] = (int)acc.size();
                acc.push_back(0);
                child.resize(acc.size() * 256, -1);
            }
            s = (unsigned)child[s * 256 + w[k]];
        }
        if (!acc[s]) acc[s] = (unsigned char)(d + 1);
    }
    const unsigned nstates = (unsigned)acc.size();
    if (nstates > MAX_TRIE) return -E2BIG;
    const unsigned nt = nstates + ndict;   // + one emission state per word
    unsigned nsp = nt;
    while (nsp % 4u != 2u) nsp++;
    const size_t need = tables_bytes(nsp, ncol);
    if (used) *used = need;
    if (!out || need > cap) return -ENOSPC;
    ScanTables* T = (ScanTables*)out;
    memset(T, 0, sizeof *T);
    T->ndict = ndict;
    T->npat = npat;
    T->nstates = nstates;
    T->ncol = ncol;
    T->nsp = nsp;
    T->emit2 = 2u * nstates;
    unsigned short* dfa = (unsigned short*)((unsigned char*)out + sizeof(ScanTables));
    for (unsigned c = 0; c < ncol; c++) {
        unsigned b;   // a byte of the column
        if (ncol == NCOL_NARROW) b = c == 0 ? 0u : (c == NCOL_NARROW - 1 ? 255u : c + 47u);
        else b = c == 128u ? 255u : c;
        for (unsigned s = 0; s < nsp; s++) {
            unsigned next = ROOT;
            if (s < nt) {
                const unsigned r = s >= nstates ? ROOT : s;   // emission states behave as ROOT
                if (!is_word_byte(b)) next = (r >= 2 && acc[r]) ? nstates + acc[r] - 1u : ROOT;
                else if (r == DEAD) next = DEAD;
                else next = child[r * 256 + b] >= 0 ? (unsigned)child[r * 256 + b] : DEAD;
            }
            dfa[(size_t)c * nsp + s] = (unsigned short)(2u * next);
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
