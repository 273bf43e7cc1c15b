// scan_emul.cu -- host-side emulation of the CUDA scan (same scan_core.cuh source as the sm_100a
// kernels), so the CPU test suite can check the kernel's scan logic against the oracle without a
// GPU.  Bytes past the end of the text are filled with word characters ('a') so that a masking
// bug would change the counts.
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <vector>

#include "scan_core.cuh"
#include "tokscan.cuh"

using namespace gsys_scan;

template <bool WIDE>
static int run(const uint8_t* text, uint64_t n, uint32_t chunk, const std::vector<uint4>& tab, uint64_t* hist,
               uint32_t npat, bool lanes, bool* any_out) {
    const ScanTables& T = *reinterpret_cast<const ScanTables*>(tab.data());
    const Dfa<WIDE> D = dfa_view<WIDE>(T);
    std::vector<uint8_t> buf(n + 96, 'a');
    if (n) memcpy(buf.data(), text, n);
    bool any = false;
    const unsigned emit2 = T.emit2;
    auto emit = [hist, emit2](unsigned e) { if (e >= emit2) hist[(e - emit2) >> 1]++; };
    auto emit2x = [hist, emit2](unsigned hi, unsigned lo) {
        if (hi >= emit2) hist[(hi - emit2) >> 1]++;
        if (lo >= emit2) hist[(lo - emit2) >> 1]++;
    };
    const long long N = (long long)n;
    for (uint64_t s = 0; s < n; s += chunk) {
        const uint64_t e = s + chunk < n ? s + chunk : n;
        const long long E = (long long)e;
        const bool grep_on = npat > 0;
        if (lanes) {   // 64-byte lane spans exactly as the kernels run them
            for (uint64_t p0 = s; p0 < e; p0 += 64) {
                uint4 V[5];
                for (int k = 0; k < 5; k++) {
                    const uint64_t q = p0 + 16 * k;
                    // past the data: the 'a' fill (the kernel zero-fills; masking must not care)
                    if (q < n) memcpy(&V[k], &buf[q], 16);
                    else V[k] = make_uint4(0, 0, 0, 0);
                }
                Win W{V[0], V[1], V[2], V[3], V[4]};
                const unsigned prevb = p0 > 0 ? buf[p0 - 1] : 0u;
                dfa_lane64(D, W, prevb, (long long)p0, E, N, emit, emit2x);
                if (grep_on && !any && grep_lane64(T, W, (long long)p0, E, N)) any = true;
            }
            continue;
        }
        for (uint64_t p0 = s; p0 < e; p0 += 16) {   // reference composition: 16-byte steps
            uint4 A, B = make_uint4(0, 0, 0, 0);
            memcpy(&A, &buf[p0], 16);
            if (p0 + 16 < n) memcpy(&B, &buf[p0 + 16], 16);
            const unsigned prevb = p0 > 0 ? buf[p0 - 1] : 0u;
            if (scan_step(T, D, A, B, prevb, (long long)p0, E, N, grep_on && !any, emit)) any = true;
        }
    }
    *any_out = any;
    return 0;
}

// Warp-cooperative token scan (tokscan.cuh tokw_*) exactly as scan_range_tokw runs it: per 2 KiB
// warp tile from each chunk start, the 32 lane spans staged in 80-byte slots, every lane's word
// masks, the next lane's first 32 mask bits as lookahead (lane 31: the 16 staged bytes after the
// tile), phase A lists the starts of all lanes in lane order, phase C looks every entry up.
static int run_tokw(const uint8_t* text, uint64_t n, uint32_t chunk, const gsys_tok::TokTables& T, uint64_t* hist,
                    uint32_t npat, bool* any_out) {
    bool any = false;
    const long long N = (long long)n;
    const gsys_tok::TokRegs R = gsys_tok::tok_regs(T);
    std::vector<uint8_t> tile(gsys_tok::TOKW_TILE, 0);
    auto byte_at = [&](long long q) -> uint8_t { return (q >= 0 && q < N) ? text[q] : 0; };
    for (uint64_t s = 0; s < n; s += chunk) {
        const long long e = (long long)(s + chunk < n ? s + chunk : n);
        for (long long base = (long long)s; base < e; base += 2048) {
            Win W[32];
            unsigned m0[32], m1[32], m2[32];
            for (unsigned l = 0; l < 32; l++) {
                const long long p0 = base + 64ll * l;
                for (unsigned i = 0; i < gsys_tok::TOKW_SLOT; i++) tile[l * gsys_tok::TOKW_SLOT + i] = byte_at(p0 + i);
                uint4 V[5];
                for (int k = 0; k < 5; k++) memcpy(&V[k], &tile[l * gsys_tok::TOKW_SLOT + 16 * k], 16);
                W[l] = Win{V[0], V[1], V[2], V[3], V[4]};
                m0[l] = gsys_tok::mask16(V[0]) | (gsys_tok::mask16(V[1]) << 16);
                m1[l] = gsys_tok::mask16(V[2]) | (gsys_tok::mask16(V[3]) << 16);
            }
            for (unsigned l = 0; l < 32; l++) m2[l] = l < 31 ? m0[l + 1] : gsys_tok::mask16(W[31].w4);
            std::vector<unsigned> list;
            for (unsigned l = 0; l < 32; l++) {
                const long long p0 = base + 64ll * l;
                const bool pw = l ? ((m1[l - 1] >> 31) & 1u) : (p0 > 0 && is_word_byte(byte_at(p0 - 1)));
                const gsys_tok::TokwSpan sp = gsys_tok::tokw_span(m0[l], m1[l], m2[l], pw, p0, e, N);
                gsys_tok::tokw_list(R, sp, l * gsys_tok::TOKW_SLOT, [&list](unsigned x) { list.push_back(x); });
                if (npat && !any && p0 < e && grep_lane64(T.g, W[l], p0, e, N)) any = true;
            }
            if (list.size() > gsys_tok::TOKW_LIST) return -E2BIG;
            const gsys_tok::TokwTile t{tile.data(), 0u};
            for (unsigned x : list) gsys_tok::tokw_lookup(T, R, t, x, [hist](unsigned d) { hist[d]++; });
        }
    }
    *any_out = any;
    return 0;
}

// mode 0: 16-byte reference steps, narrow table; 1: 64-byte lane spans, narrow table (wc_kernel);
// 2: 64-byte lane spans, wide table (scan_kernel); 3: 16-byte reference steps, wide table;
// 4: warp-cooperative token scan (tokscan.cuh tokw_*).
extern "C" int scan_emul2(const uint8_t* text, uint64_t n, uint32_t chunk, const char* dict, const uint8_t* dlen,
                          uint32_t ndict, const char* pats, const uint8_t* plen, uint32_t npat, uint64_t* hist,
                          uint32_t* hit, int mode) {
    if (chunk < 16 || chunk % 16 || mode < 0 || mode > 4) return -EINVAL;
    if (mode == 4) {
        std::vector<uint4> tt((sizeof(gsys_tok::TokTables) + 15) / 16);
        int rc = gsys_tok::build_tok_tables(tt.data(), tt.size() * 16, dict, dlen, ndict, pats, plen, npat, nullptr);
        if (rc) return rc;
        bool any = false;
        const auto& TT = *reinterpret_cast<const gsys_tok::TokTables*>(tt.data());
        rc = run_tokw(text, n, chunk, TT, hist, npat, &any);
        if (hit) *hit = any ? 1u : 0u;
        return rc;
    }
    const bool wide = mode >= 2;
    const unsigned ncol = wide ? NCOL_WIDE : NCOL_NARROW;
    size_t tb = 0;
    int rc = build_tables(nullptr, 0, dict, dlen, ndict, pats, plen, npat, &tb, ncol);
    if (rc && rc != -ENOSPC) return rc;
    std::vector<uint4> tab((tb + 15) / 16);
    rc = build_tables(tab.data(), tab.size() * 16, dict, dlen, ndict, pats, plen, npat, nullptr, ncol);
    if (rc) return rc;
    bool any = false;
    const bool lanes = mode == 1 || mode == 2;
    rc = wide ? run<true>(text, n, chunk, tab, hist, npat, lanes, &any) : run<false>(text, n, chunk, tab, hist, npat, lanes, &any);
    if (hit) *hit = any ? 1u : 0u;
    return rc;
}

extern "C" int scan_emul(const uint8_t* text, uint64_t n, uint32_t chunk, const char* dict, const uint8_t* dlen,
                         uint32_t ndict, const char* pats, const uint8_t* plen, uint32_t npat, uint64_t* hist,
                         uint32_t* hit) {
    return scan_emul2(text, n, chunk, dict, dlen, ndict, pats, plen, npat, hist, hit, 0);
}
