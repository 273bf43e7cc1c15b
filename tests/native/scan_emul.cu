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

extern "C" int scan_emul(const uint8_t* text, uint64_t n, uint32_t chunk, const char* dict, const uint8_t* dlen,
                         uint32_t ndict, const char* pats, const uint8_t* plen, uint32_t npat, uint64_t* hist,
                         uint32_t* hit) {
    if (chunk < 16 || chunk % 16) return -EINVAL;
    ScanTables T;
    int rc = build_tables(&T, dict, dlen, ndict, pats, plen, npat);
    if (rc) return rc;
    std::vector<uint8_t> buf(n + 64, 'a');
    if (n) memcpy(buf.data(), text, n);
    bool any = false;
    for (uint64_t s = 0; s < n; s += chunk) {
        uint64_t e = s + chunk < n ? s + chunk : n;
        bool grep_on = npat > 0;
        for (uint64_t p0 = s; p0 < e; p0 += 16) {
            uint4 A, B;
            memcpy(&A, &buf[p0], 16);
            if (p0 + 16 < n) memcpy(&B, &buf[p0 + 16], 16);
            else B = make_uint4(0, 0, 0, 0);
            unsigned prevb = p0 > 0 ? buf[p0 - 1] : 0u;
            bool h = scan_step(T, A, B, prevb, (long long)p0, (long long)e, (long long)n, grep_on && !any,
                               [hist](unsigned d) { hist[d]++; });
            if (h) any = true;
        }
    }
    if (hit) *hit = any ? 1u : 0u;
    return 0;
}
