// tokscan.cuh -- token-level wordcount step (row a8, SURVEY.md sec. 8a "SWAR token starts ->
// length filter -> verify against the dictionary"), shared by the sm_100a kernels
// (gsys_kernels.cu) and the host emulation used by CPU tests (tests/native/scan_emul.cu).  Part of
// the CUDA path: the oracle (oracle/) never includes it.
//
// Same definitions as scan_core.cuh (reading A9/A10): a token is a maximal run of [A-Za-z0-9_],
// owned by the chunk holding its first byte; a dictionary hit is a whole token byte-equal to one
// of <= 64 words of <= 16 bytes ("search for occurrences of 64 strings", PAPER.md:32 P32.6).
//
// Instead of one DFA lookup per byte (scan_core.cuh: a dependent shared-memory gather per byte), a
// warp classifies each lane's 64-byte span four bytes per SWAR step into word-byte masks, lists the
// token starts of the whole 2 KiB tile (offset + length from the masks), and then looks the listed
// tokens up with every lane taking every 32nd entry: the token's first 16 bytes (aligned shared
// loads + funnel shifts), masked to its length, hashed into a collision-free table of the dictionary
// (the builder picks multipliers until the words land in distinct slots), verified byte-exactly
// against the slot's key.  Measured against the DFA in DESIGN.md sec. 6.
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
    uint4 nokey;                // all 0xff: the "key" of an empty slot (no masked token equals it);
                                // it sits right before key[0], so slot value id reads key[id - 1]
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

// word4() plus grep's first-byte prefilter on the same 7-bit byte values (grep_lane64's SWAR
// range test, fused: two IMADs and one LOP3 more per 4 bytes); gacc collects bit 7 of every byte
// whose low 7 bits fall in the patterns' first-byte range.
GSYS_HD unsigned word4g(unsigned w, unsigned one, unsigned add_lo, unsigned add_hi, unsigned& gacc) {
    const unsigned a = w & 0x7f7f7f7fu;
    gacc |= (a * one + add_lo) & ~(a * one + add_hi);
    const unsigned x = a | 0x20202020u;
    const unsigned g1 = x * one + 0x1f1f1f1fu;
    const unsigned g2 = x * one + 0x05050505u;
    const unsigned g3 = a * one + 0x50505050u;
    const unsigned g4 = a * one + 0x46464646u;
    const unsigned nu = (a ^ 0x5f5f5f5fu) * one + 0x7f7f7f7fu;
    const unsigned v = (g1 & ~g2) | (g3 & ~g4);
    return (v | ~nu) & ~w & 0x80808080u;
}
GSYS_HD unsigned mask16g(const uint4& q, unsigned one, unsigned add_lo, unsigned add_hi, unsigned& gacc) {
    return pack16(word4g(q.x, one, add_lo, add_hi, gacc), word4g(q.y, one, add_lo, add_hi, gacc),
                  word4g(q.z, one, add_lo, add_hi, gacc), word4g(q.w, one, add_lo, add_hi, gacc));
}

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
    return v;   // ld.u8 into a 32-bit register zero-extends
#else
    (void)R;
    return T.slot[h];
#endif
}
// ------------------------------------------------------------------ warp-cooperative token scan
// Round-2 form of the token path.  The first version ran each lane's tokens in a
// lane-serial loop, so a warp spent as many rounds as its busiest lane had tokens (1.5-1.7x the
// mean) on ~130-instruction iterations.  Here a warp tile is handled in two phases:
//   A  every lane lists the token starts of its 64-byte span -- one u16 entry per start: the
//      token's byte offset in the staged tile and its length (a few instructions per token);
//   C  the warp's list is looked up with lane j taking entries j, j+32, ... (even work per lane):
//      5 aligned shared loads + 4 funnel shifts give the first 16 bytes, a multiply hash of the
//      first 8 and the length picks the dictionary slot, one 16-byte key load (predicated: only
//      lanes whose slot is taken) verifies the whole token.
// Entry: bits 0..11 = offset in the staged tile (lane * TOKW_SLOT + q), bits 12..15 = length - 1;
// TOKW_SKIP for a start no dictionary word can match (length > 16 or not in lenmask).  TOKW_SKIP
// decodes like an entry (offset 32 * TOKW_SLOT, the tile's tail area -- inside the staging buffer,
// which holds TOKW_TILE bytes -- length 1), so phase C runs it through the same straight-line
// lookup and only its final emit is gated off.
constexpr unsigned TOKW_SLOT = 80;          // staged lane slot: the 64 span bytes + the 16 after them
constexpr unsigned TOKW_SKIP = 32u * TOKW_SLOT;
constexpr unsigned TOKW_TILE = 32u * TOKW_SLOT + 32u;   // a staged tile: slots, the 4 bytes before it, guard
constexpr unsigned TOKW_LIST = 1024;        // entries per warp tile (at most one start per 2 bytes)

// The owned token starts of one lane span and its word-byte masks.  m0, m1: bytes 0..31, 32..63 of
// the span; m2: the 32 bytes after it (at least the first 16 exact); prev_word: byte p0-1 exists
// and is a word byte.  Bytes at or past valid_end never belong to a token; starts at or past
// own_end are not owned.
struct TokwSpan {
    unsigned s0, s1;        // starts among bytes 0..31 / 32..63
    unsigned m0, m1, m2;
};
GSYS_HD TokwSpan tokw_span(unsigned m0, unsigned m1, unsigned m2, bool prev_word, long long p0, long long own_end,
                           long long valid_end) {
    const long long nvalid_ll = valid_end - p0;
    if (nvalid_ll < 96) {
        const unsigned nv = nvalid_ll <= 0 ? 0u : (unsigned)nvalid_ll;
        m0 &= nv >= 32u ? ~0u : ((1u << nv) - 1u);
        m1 &= nv >= 64u ? ~0u : (nv <= 32u ? 0u : ((1u << (nv - 32u)) - 1u));
        m2 &= nv <= 64u ? 0u : ((1u << (nv - 64u)) - 1u);
    }
    TokwSpan r;
    r.m0 = m0;
    r.m1 = m1;
    r.m2 = m2;
    r.s0 = m0 & ~((m0 << 1) | (prev_word ? 1u : 0u));
    r.s1 = m1 & ~((m1 << 1) | (m0 >> 31));
    const long long nown_ll = own_end - p0;
    if (nown_ll < 64) {
        const unsigned no = nown_ll <= 0 ? 0u : (unsigned)nown_ll;
        r.s0 &= no >= 32u ? ~0u : ((1u << no) - 1u);
        r.s1 &= no <= 32u ? 0u : ((1u << (no - 32u)) - 1u);
    }
    return r;
}

GSYS_HD unsigned tokw_brev(unsigned x) {
#ifdef __CUDA_ARCH__
    return __brev(x);
#else
    x = ((x >> 1) & 0x55555555u) | ((x & 0x55555555u) << 1);
    x = ((x >> 2) & 0x33333333u) | ((x & 0x33333333u) << 2);
    x = ((x >> 4) & 0x0f0f0f0fu) | ((x & 0x0f0f0f0fu) << 4);
    x = ((x >> 8) & 0x00ff00ffu) | ((x & 0x00ff00ffu) << 8);
    return (x >> 16) | (x << 16);
#endif
}
GSYS_HD unsigned tokw_fshl(unsigned lo, unsigned hi, unsigned sh) {   // upper 32 bits of (hi:lo) << (sh & 31)
#ifdef __CUDA_ARCH__
    return __funnelshift_l(lo, hi, sh);
#else
    sh &= 31u;
    return sh ? (hi << sh) | (lo >> (32u - sh)) : hi;
#endif
}

// Position of the highest set bit (x != 0): one FLO (PTX bfind).
GSYS_HD unsigned tokw_hibit(unsigned x) {
#ifdef __CUDA_ARCH__
    unsigned r;
    asm("bfind.u32 %0, %1;" : "=r"(r) : "r"(x));
    return r;
#else
    return 31u - (unsigned)__builtin_clz(x);
#endif
}

// Phase A: one entry per start of the span; put(entry) appends it.  slot_off = the span's offset
// in the staged tile.  Starts are taken highest first (one FLO each); the token length comes from
// the bit-reversed 64-bit window of the mask as a count of leading ones: p = the highest 0 of the
// shifted window (a guard bit at 14 caps the count at 17), len = 31 - p.  lenrev is lenmask
// reversed (bit 31 - L for length L), so it is tested at p directly.
template <class Put>
GSYS_HD void tokw_list(const TokRegs& R, const TokwSpan& sp, unsigned slot_off, Put&& put) {
    const unsigned lenrev = tokw_brev(R.lenmask);
GSYS_UNROLL
    for (int h = 0; h < 2; h++) {
        unsigned S = h ? sp.s1 : sp.s0;
        const unsigned lo = h ? sp.m1 : sp.m0, hi = h ? sp.m2 : sp.m1;
        const unsigned ylo = tokw_brev(hi), yhi = tokw_brev(lo);   // the 64-bit window reversed
        // entry = (slot_off + 32h + q) | ((len - 1) << 12) = base + q - (p << 12), len = 31 - p
        const unsigned base = slot_off + 32u * (unsigned)h + (30u << 12);
        while (S) {
            const unsigned q = tokw_hibit(S);
            S ^= 1u << q;
            const unsigned z = tokw_fshl(ylo, yhi, q);        // bit 31 - k = mask bit q + k
            const unsigned p = tokw_hibit(~z | 0x4000u);      // 31 - (run of word bytes from q), run <= 17
            put(((lenrev >> p) & 1u) ? base + q - (p << 12) : TOKW_SKIP);
        }
    }
}

// The staged tile: a pointer (host emulation) and its shared-window address (device).
struct TokwTile {
    const unsigned char* p;
    unsigned s;
};
GSYS_HD unsigned tokw_ld32(const TokwTile& t, unsigned off) {   // off: 4-byte aligned
#ifdef __CUDA_ARCH__
    // not volatile: the address depends on a list entry loaded after the warp's barrier, and the
    // staged bytes do not change during the lookups, so the compiler may interleave two lookups
    unsigned v;
    asm("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(t.s + off));
    return v;
#else
    unsigned v;
    memcpy(&v, t.p + off, 4);
    return v;
#endif
}
// Phase C: look up one entry; emit(d) counts a hit of word d.  Straight-line: the 16 bytes at the
// token start (5 aligned loads, 4 funnel shifts), masked to the token's length; the slot of
// (first 8 bytes, length); the slot's key (an empty slot reads `nokey`, which equals no token);
// a hit is all 16 bytes equal -- keys are zero-padded and word bytes are never 0, so equal masked
// bytes mean equal lengths too.
template <class Emit>
GSYS_HD void tokw_lookup(const TokTables& T, const TokRegs& R, const TokwTile& tile, unsigned e, Emit&& emit) {
    const unsigned off = e & 0xfffu, len = (e >> 12) + 1u;
    const unsigned a4 = off & ~3u;
    const unsigned sh = off * 8u;   // funnel shifts take the amount mod 32
    const unsigned w0 = tokw_ld32(tile, a4), w1 = tokw_ld32(tile, a4 + 4u), w2 = tokw_ld32(tile, a4 + 8u);
    const unsigned w3 = tokw_ld32(tile, a4 + 12u), w4 = tokw_ld32(tile, a4 + 16u);
    // bytes 0..len-1 kept: two 64-bit shifts (PTX clamps shift amounts at the width); ALU work
    // instead of a mask-table load -- the lookups are bound by the shared-memory pipe
    const unsigned n8 = 8u * len, m8 = n8 > 64u ? n8 - 64u : 0u;
    unsigned long long k0, k1;
#ifdef __CUDA_ARCH__
    asm("shl.b64 %0, %1, %2;" : "=l"(k0) : "l"(~0ull), "r"(n8));
    asm("shl.b64 %0, %1, %2;" : "=l"(k1) : "l"(~0ull), "r"(m8));
#else
    k0 = n8 >= 64u ? 0ull : (~0ull << n8);
    k1 = m8 >= 64u ? 0ull : (~0ull << m8);
#endif
    const unsigned a = GSYS_FSHR(w0, w1, sh) & ~(unsigned)k0, b = GSYS_FSHR(w1, w2, sh) & ~(unsigned)(k0 >> 32);
    const unsigned c = GSYS_FSHR(w2, w3, sh) & ~(unsigned)k1, d = GSYS_FSHR(w3, w4, sh) & ~(unsigned)(k1 >> 32);
    const unsigned id = tok_slot(T, R, ((a * R.m0) ^ (b * R.m1) ^ (len * R.m4)) >> (32u - HBITS));
    // the slot's key, loaded only by lanes whose slot is taken (a predicated load: no branch, and
    // lanes with an empty slot add no shared-memory wavefronts); an empty slot keeps `nokey`
    uint4 k = make_uint4(0xffffffffu, 0xffffffffu, 0xffffffffu, 0xffffffffu);
#ifdef __CUDA_ARCH__
    asm("{ .reg .pred p; setp.ne.u32 p, %4, 0;\n\t"
        "@p ld.shared.v4.u32 {%0, %1, %2, %3}, [%5]; }"
        : "+r"(k.x), "+r"(k.y), "+r"(k.z), "+r"(k.w)
        : "r"(id), "r"(R.tabs + (unsigned)offsetof(TokTables, nokey) + 16u * id));
#else
    if (id) k = T.key[id - 1u];
#endif
    if (((a ^ k.x) | (b ^ k.y) | (c ^ k.z) | (d ^ k.w)) == 0u && e != TOKW_SKIP) emit(id - 1u);
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
    memset(&T->nokey, 0xff, sizeof T->nokey);
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
