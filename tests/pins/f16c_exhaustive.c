/* Pin for the oracle's bit-level fp32 -> fp16 RNE conversion: compare it with the host
 * CPU's F16C instruction (vcvtps2ph, round-to-nearest-even, IEEE subnormals) over ALL
 * 2^32 fp32 bit patterns.  NaNs compare by class (both NaN).  Prints the mismatch count.
 * Test infrastructure; links ../../oracle/liboracle.so.  Built by tests/test_oracle_split.py. */
#include <immintrin.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>

uint16_t oracle_f32_to_f16_rne(uint32_t x);
uint32_t oracle_f16_to_f32(uint16_t h);

static int is_nan16(uint16_t h) { return ((h & 0x7c00u) == 0x7c00u) && (h & 0x3ffu); }

int main(void)
{
    long long bad = 0, bad_back = 0;
#pragma omp parallel for reduction(+ : bad, bad_back) schedule(static)
    for (long long hiw = 0; hiw < 65536; hiw++) {
        for (uint32_t low = 0; low < 65536; low += 8) {
            uint32_t u[8];
            for (int t = 0; t < 8; t++) u[t] = ((uint32_t)hiw << 16) | (low + t);
            __m256 v;
            memcpy(&v, u, 32);
            __m128i h = _mm256_cvtps_ph(v, _MM_FROUND_TO_NEAREST_INT | _MM_FROUND_NO_EXC);
            uint16_t hw[8];
            memcpy(hw, &h, 16);
            for (int t = 0; t < 8; t++) {
                uint16_t o = oracle_f32_to_f16_rne(u[t]);
                if (o != hw[t] && !(is_nan16(o) && is_nan16(hw[t]))) bad++;
            }
        }
        /* fp16 -> fp32 decode vs vcvtph2ps, all 65536 patterns (once, by hiw == 0) */
        if (hiw == 0) {
            for (uint32_t p = 0; p < 65536; p += 8) {
                uint16_t hh[8];
                for (int t = 0; t < 8; t++) hh[t] = (uint16_t)(p + t);
                __m128i hv;
                memcpy(&hv, hh, 16);
                __m256 f = _mm256_cvtph_ps(hv);
                uint32_t fu[8];
                memcpy(fu, &f, 32);
                for (int t = 0; t < 8; t++) {
                    uint32_t o = oracle_f16_to_f32(hh[t]);
                    int on = ((o & 0x7f800000u) == 0x7f800000u) && (o & 0x7fffffu);
                    int hn = ((fu[t] & 0x7f800000u) == 0x7f800000u) && (fu[t] & 0x7fffffu);
                    if (o != fu[t] && !(on && hn)) bad_back++;
                }
            }
        }
    }
    printf("%lld %lld\n", bad, bad_back);
    return 0;
}
