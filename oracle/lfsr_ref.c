/*
 * oracle/lfsr_ref.c -- bit-serial Fibonacci LFSR reference (CPU, plain C99).
 *
 * TEST INFRASTRUCTURE ONLY (see oracle/mickey2_ref.c for the rule).
 *
 * PAPER.md:545-596 (sec. 4.3, Eq. 2, Figs. 7-8): the bitsliced LFSR -- an
 * n-bit shift register with feedback polynomial g(x) = sum a_i x^i over GF(2),
 * k = |{a_i != 0}| feedback taps, one output bit per shift
 * (Eq. 1): a primitive polynomial gives period 2^n - 1.  The paper fixes no
 * particular polynomial; reading L1 takes n = 128 and the
 * primitive p(x) = x^128 + x^29 + x^27 + x^2 + 1 in Fibonacci form:
 *     s_{t+128} = s_{t+29} + s_{t+27} + s_{t+2} + s_t,   output z_t = s_t,
 * initial state s_0..s_127 = the 16 key bytes, MSB-first; keystream packed
 * MSB-first.
 *
 * Pins (tests/test_oracle_lfsr.py): the step matrix driven through this code
 * has order exactly 2^128 - 1, and Berlekamp-Massey recovers exactly p(x)
 * (linear complexity 128) from its output.
 */
#include <stdint.h>
#include <string.h>

#define L_N 128

static int clock_lfsr(uint8_t s[L_N])
{
    const int z = s[0];
    const uint8_t fb = (uint8_t)(s[29] ^ s[27] ^ s[2] ^ s[0]);
    memmove(s, s + 1, L_N - 1);
    s[L_N - 1] = fb;
    return z;
}

void ref_lfsr128_keystream(const uint8_t key[16], uint64_t nbits, uint8_t* out)
{
    uint8_t s[L_N];
    uint64_t t;
    int i;
    for (i = 0; i < L_N; i++) s[i] = (uint8_t)((key[i / 8] >> (7 - i % 8)) & 1);
    memset(out, 0, (size_t)((nbits + 7) / 8));
    for (t = 0; t < nbits; t++) out[t / 8] |= (uint8_t)(clock_lfsr(s) << (7 - t % 8));
}

/* one shift on an explicit state (0/1 bytes), returns the output bit */
int ref_lfsr128_clock(uint8_t* s) { return clock_lfsr(s); }
