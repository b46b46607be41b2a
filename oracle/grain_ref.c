/*
 * oracle/grain_ref.c -- bit-serial Grain v1 reference (CPU, plain C99).
 *
 * TEST INFRASTRUCTURE ONLY (see oracle/mickey2_ref.c for the rule): only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference legs
 * may load it; it shares nothing with the CUDA path.
 *
 * PAPER.md:339-357 (sec. 2.3.3, Fig. 4): Grain, eSTREAM profile 2 -- an 80-bit
 * LFSR and an 80-bit NFSR, functions f (LFSR feedback), g (NFSR feedback) and
 * the filter h; 80-bit key, 64-bit IV, 160 initialisation clocks.  The paper
 * defers the definition to ref [15]; below is that
 * specification written out in its own notation and order (DESIGN.md readings
 * G1-G3).  Registers are arrays of bits; one clock = one output bit.
 *
 * Pins (tests/test_oracle_grain.py): the specification's two test vectors,
 * LFSR primitivity (period 2^80 - 1), bit-flip wiring of f / g / h / z.
 */
#include <stdint.h>
#include <string.h>

#define GR_LEN 80

typedef struct {
    uint8_t s[GR_LEN]; /* LFSR s_i .. s_{i+79} */
    uint8_t b[GR_LEN]; /* NFSR b_i .. b_{i+79} */
} gr_state;

/* f: s_{i+80} = s_{i+62} + s_{i+51} + s_{i+38} + s_{i+23} + s_{i+13} + s_i */
static int f_lfsr(const gr_state* st)
{
    const uint8_t* s = st->s;
    return s[62] ^ s[51] ^ s[38] ^ s[23] ^ s[13] ^ s[0];
}

/* g: b_{i+80} = s_i + (the NFSR feedback polynomial g over b) */
static int g_nfsr(const gr_state* st)
{
    const uint8_t* b = st->b;
    return st->s[0] ^ b[62] ^ b[60] ^ b[52] ^ b[45] ^ b[37] ^ b[33] ^ b[28] ^ b[21] ^ b[14] ^ b[9] ^ b[0] ^
           (b[63] & b[60]) ^ (b[37] & b[33]) ^ (b[15] & b[9]) ^ (b[60] & b[52] & b[45]) ^
           (b[33] & b[28] & b[21]) ^ (b[63] & b[45] & b[28] & b[9]) ^ (b[60] & b[52] & b[37] & b[33]) ^
           (b[63] & b[60] & b[21] & b[15]) ^ (b[63] & b[60] & b[52] & b[45] & b[37]) ^
           (b[33] & b[28] & b[21] & b[15] & b[9]) ^ (b[52] & b[45] & b[37] & b[33] & b[28] & b[21]);
}

/* h(x0..x4), x0 = s_{i+3}, x1 = s_{i+25}, x2 = s_{i+46}, x3 = s_{i+64}, x4 = b_{i+63} */
static int h_filter(const gr_state* st)
{
    const int x0 = st->s[3], x1 = st->s[25], x2 = st->s[46], x3 = st->s[64], x4 = st->b[63];
    return x1 ^ x4 ^ (x0 & x3) ^ (x2 & x3) ^ (x3 & x4) ^ (x0 & x1 & x2) ^ (x0 & x2 & x3) ^ (x0 & x2 & x4) ^
           (x1 & x2 & x4) ^ (x2 & x3 & x4);
}

/* z_i = sum_{k in A} b_{i+k} + h, A = {1, 2, 4, 10, 31, 43, 56} */
static int output_bit(const gr_state* st)
{
    const uint8_t* b = st->b;
    return b[1] ^ b[2] ^ b[4] ^ b[10] ^ b[31] ^ b[43] ^ b[56] ^ h_filter(st);
}

/* One clock; `init` = the initialisation mode where z is fed back into both
 * registers.  Returns the z produced before the shift. */
static int clock_grain(gr_state* st, int init)
{
    const int z = output_bit(st);
    int fs = f_lfsr(st), fb = g_nfsr(st);
    if (init) {
        fs ^= z;
        fb ^= z;
    }
    memmove(st->s, st->s + 1, GR_LEN - 1);
    memmove(st->b, st->b + 1, GR_LEN - 1);
    st->s[GR_LEN - 1] = (uint8_t)fs;
    st->b[GR_LEN - 1] = (uint8_t)fb;
    return z;
}

/* bit i of a byte string, LSB-first (reading G2) */
static int lsb_bit(const uint8_t* buf, int i) { return (buf[i / 8] >> (i % 8)) & 1; }

static void init(gr_state* st, const uint8_t key[10], const uint8_t iv[8])
{
    int i;
    for (i = 0; i < 80; i++) st->b[i] = (uint8_t)lsb_bit(key, i);
    for (i = 0; i < 64; i++) st->s[i] = (uint8_t)lsb_bit(iv, i);
    for (i = 64; i < 80; i++) st->s[i] = 1;
    for (i = 0; i < 160; i++) clock_grain(st, 1);
}

/* Keystream of one instance: nbits bits packed LSB-first into out. */
void ref_grain_keystream(const uint8_t key[10], const uint8_t iv[8], uint64_t nbits, uint8_t* out)
{
    gr_state st;
    uint64_t t;
    init(&st, key, iv);
    memset(out, 0, (size_t)((nbits + 7) / 8));
    for (t = 0; t < nbits; t++) out[t / 8] |= (uint8_t)(clock_grain(&st, 0) << (t % 8));
}

/* State after init plus extra keystream clocks: s_out[i] = s_i, b_out[i] = b_i. */
void ref_grain_state(const uint8_t key[10], const uint8_t iv[8], uint64_t extra_clocks, uint8_t* s_out,
                     uint8_t* b_out)
{
    gr_state st;
    uint64_t t;
    init(&st, key, iv);
    for (t = 0; t < extra_clocks; t++) clock_grain(&st, 0);
    memcpy(s_out, st.s, GR_LEN);
    memcpy(b_out, st.b, GR_LEN);
}

/* One clock on an explicit state (for the wiring tests); returns z. */
int ref_grain_clock(uint8_t* s, uint8_t* b, int init_mode)
{
    gr_state st;
    int z;
    memcpy(st.s, s, GR_LEN);
    memcpy(st.b, b, GR_LEN);
    z = clock_grain(&st, init_mode);
    memcpy(s, st.s, GR_LEN);
    memcpy(b, st.b, GR_LEN);
    return z;
}
