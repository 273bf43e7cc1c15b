// scan_emul.cu -- host-side emulation of the CUDA scan (same scan_core.cuh source as the sm_100a
// kernels), so the CPU test suite can check the kernel's scan logic against the oracle without a
// GPU.  Bytes past the end of the text are filled with word characters ('a') so that a masking
// bug would change the counts.
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <vector>

#include "scan_core.cuh"

using namespace gsys_scan;

// pairs = 0: every 16-byte step through scan_step (reference composition);
// pairs = 1: steps taken two at a time through dfa_pair + dfa_finish exactly as the kernels do
// (falling back to dfa_segment when either step is not full), grep through grep_step.
extern "C" int scan_emul2(const uint8_t* text, uint64_t n, uint32_t chunk, const char* dict, const uint8_t* dlen,
                          uint32_t ndict, const char* pats, const uint8_t* plen, uint32_t npat, uint64_t* hist,
                          uint32_t* hit, int pairs) {
    if (chunk < 16 || chunk % 16) return -EINVAL;
    size_t tb = 0;
    int rc = build_tables(nullptr, 0, dict, dlen, ndict, pats, plen, npat, &tb);
    if (rc && rc != -ENOSPC) return rc;
    std::vector<uint4> tab((tb + 15) / 16);
    rc = build_tables(tab.data(), tab.size() * 16, dict, dlen, ndict, pats, plen, npat, nullptr);
    if (rc) return rc;
    const ScanTables& T = *reinterpret_cast<const ScanTables*>(tab.data());
    const unsigned short* dfa = reinterpret_cast<const unsigned short*>(
        reinterpret_cast<const unsigned char*>(tab.data()) + sizeof(ScanTables));
    std::vector<uint8_t> buf(n + 64, 'a');
    if (n) memcpy(buf.data(), text, n);
    bool any = false;
    for (uint64_t s = 0; s < n; s += chunk) {
        uint64_t e = s + chunk < n ? s + chunk : n;
        bool grep_on = npat > 0;
        auto on_hit = [hist](unsigned h) { if (h) hist[h - 1]++; };
        auto load = [&](uint64_t p0, uint4& A, uint4& B, unsigned& prevb) {
            memcpy(&A, &buf[p0], 16);
            if (p0 + 16 < n) memcpy(&B, &buf[p0 + 16], 16);
            else B = make_uint4(0, 0, 0, 0);
            prevb = p0 > 0 ? buf[p0 - 1] : 0u;
        };
        const long long E = (long long)e, N = (long long)n;
        if (pairs == 2) {   // 64-byte lane spans exactly as the kernels run them
            for (uint64_t p0 = s; p0 < e; p0 += 64) {
                uint4 V[5];
                for (int k = 0; k < 5; k++) {
                    uint64_t q = p0 + 16 * k;
                    if (q < n) memcpy(&V[k], &buf[q], 16);
                    else V[k] = make_uint4(0, 0, 0, 0);
                }
                Win W{V[0], V[1], V[2], V[3], V[4]};
                unsigned prevb = p0 > 0 ? buf[p0 - 1] : 0u;
                dfa_lane64(dfa, W, prevb, (long long)p0, E, N, on_hit);
                if (grep_on && !any && grep_lane64(T, W, (long long)p0, E, N)) any = true;
            }
            continue;
        }
        for (uint64_t p0 = s; p0 < e; p0 += pairs ? 32 : 16) {
            uint4 A, B;
            unsigned prevb;
            load(p0, A, B, prevb);
            if (!pairs) {
                bool h = scan_step(T, dfa, A, B, prevb, (long long)p0, E, N, grep_on && !any, on_hit);
                if (h) any = true;
                continue;
            }
            const uint64_t p1 = p0 + 16;
            uint4 A1 = make_uint4(0, 0, 0, 0), B1 = make_uint4(0, 0, 0, 0);
            unsigned prev1 = 0;
            if (p1 < e) load(p1, A1, B1, prev1);
            const bool full0 = (long long)p0 + 16 <= E && (long long)p0 + 16 <= N;
            const bool full1 = (long long)p1 + 16 <= E && (long long)p1 + 16 <= N;
            if (full0 && full1) {
                unsigned s0 = start_state(prevb, (long long)p0), s1 = start_state(prev1, (long long)p1);
                dfa_pair(dfa, s0, s1, A, A1, on_hit);
                const long long nv0 = N - (long long)p0, nv1 = N - (long long)p1;
                dfa_finish(dfa, s0, A, B, 16u, nv0 >= 32 ? 32u : (unsigned)nv0, on_hit);
                dfa_finish(dfa, s1, A1, B1, 16u, nv1 >= 32 ? 32u : (unsigned)nv1, on_hit);
            } else {
                dfa_segment(dfa, A, B, prevb, (long long)p0, E, N, on_hit);
                if (p1 < e) dfa_segment(dfa, A1, B1, prev1, (long long)p1, E, N, on_hit);
            }
            if (grep_on && !any) {
                if (grep_step(T, A, B, (long long)p0, E, N) || (p1 < e && grep_step(T, A1, B1, (long long)p1, E, N)))
                    any = true;
            }
        }
    }
    if (hit) *hit = any ? 1u : 0u;
    return 0;
}

extern "C" int scan_emul(const uint8_t* text, uint64_t n, uint32_t chunk, const char* dict, const uint8_t* dlen,
                         uint32_t ndict, const char* pats, const uint8_t* plen, uint32_t npat, uint64_t* hist,
                         uint32_t* hit) {
    return scan_emul2(text, n, chunk, dict, dlen, ndict, pats, plen, npat, hist, hit, 0);
}
