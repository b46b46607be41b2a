/*
 * oracle/mickey2_ref.c -- bit-serial MICKEY 2.0 reference (CPU, plain C99).
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this code.  The
 * product path (paper_conf_icppw_monfaredhkzrg20_b200/, include/, csrc/) never
 * includes, links or calls it, and it shares no header, table or helper with
 * the CUDA path.
 *
 * What it computes: the MICKEY 2.0 keystream of ONE (key, IV) instance, one bit
 * per clock, exactly as the cipher specification defines it.  PAPER.md does not
 * restate the cipher; it defers to the specification, ref [5]:
 *   - PAPER.md:246-257 (sec. 2.3.1): two 100-bit registers R (linear) and S
 *     (non-linear), mutually irregularly clocked; <=2^40 bits per key/IV.
 *   - PAPER.md:258-273 (Fig. 2): control bits "R 67 / S 34" and "S 67 / R 33",
 *     the mixing input into R.
 *   - PAPER.md:597-638 (sec. 4.4, Fig. 9): 80-bit IV, key K, input generator,
 *     controller bits, 1 output bit per instance per clock.
 *   - PAPER.md:870-871: ref [5], the MICKEY 2.0 specification, whose
 *     CLOCK_R / CLOCK_S / CLOCK_KG procedures and tables are written out
 *     below in the specification's own order and notation (DESIGN.md
 *     "Readings" R1-R4, R6, R10 list where the paper is silent or garbled).
 *
 * Nothing here is blocked, fused, sliced or reordered: each register is an
 * array of 100 bits (one uint8_t per bit), each procedure is a literal loop
 * over i, and the tables are the specification's bit ROWS (index 0..99,
 * written in groups of ten), never packed masks.
 *
 * Pins (tests/test_oracle_mickey2.py): spec test vectors T1/T2/T3
 * (tests/golden/mickey2_spec_vectors.txt), table invariants (|RTAPS| = 50,
 * FB-category counts), zero-state fixed point, control-bit algebra checks,
 * keystream-prefix consistency.
 */
#include <stdint.h>
#include <string.h>

#define M2_LEN 100

/* ---- Specification tables (spec [5]; rows i = 0..99) --- */

/* RTAPS: the set of feedback tap positions of register R. */
static const int RTAPS[] = {
     0,  1,  3,  4,  5,  6,  9, 12, 13, 16,
    19, 20, 21, 22, 25, 28, 37, 38, 41, 42,
    45, 46, 50, 52, 54, 56, 58, 60, 61, 63,
    64, 65, 66, 67, 71, 72, 79, 80, 81, 82,
    87, 88, 89, 90, 91, 92, 94, 95, 96, 97};
#define N_RTAPS ((int)(sizeof(RTAPS) / sizeof(RTAPS[0])))

/* COMP0 / COMP1 (used for i = 1..98), FB0 / FB1 (i = 0..99).  Character i of
 * each string is the table entry for index i. */
static const char COMP0[] =
    "0000110001" "0111101001" "0101010101" "1010010000" "0001010101"
    "0000101001" "1110010101" "1111111101" "0111111010" "1000000110";
static const char COMP1[] =
    "0101100101" "1110010100" "0110101110" "1111000110" "1011100001"
    "0001011100" "0111111010" "1110111100" "0100001110" "0010011000";
static const char FB0[] =
    "1111010111" "1111100101" "1111111110" "0110000001" "1100100101"
    "0100101111" "0101010000" "0000011010" "0011011100" "1110011000";
static const char FB1[] =
    "1110111000" "0111010011" "0001001100" "1011000110" "0000110110"
    "0010001001" "0010110101" "0010100011" "1101111100" "0000100001";

static int tbl(const char* row, int i) { return row[i] == '1'; }

typedef struct {
    uint8_t r[M2_LEN];
    uint8_t s[M2_LEN];
} m2_state;

/* CLOCK_R(R, INPUT_BIT_R, CONTROL_BIT_R) -- spec [5]. */
static void clock_r(m2_state* st, int input_bit_r, int control_bit_r)
{
    uint8_t r_new[M2_LEN];
    int feedback_bit = st->r[99] ^ input_bit_r;
    int i, t;
    /* r'_i = r_{i-1} for 1 <= i <= 99; r'_0 = 0 */
    r_new[0] = 0;
    for (i = 1; i < M2_LEN; i++) r_new[i] = st->r[i - 1];
    /* r'_i ^= FEEDBACK_BIT for i in RTAPS */
    for (t = 0; t < N_RTAPS; t++) r_new[RTAPS[t]] ^= (uint8_t)feedback_bit;
    /* if CONTROL_BIT_R: r'_i ^= r_i for all i */
    if (control_bit_r)
        for (i = 0; i < M2_LEN; i++) r_new[i] ^= st->r[i];
    memcpy(st->r, r_new, M2_LEN);
}

/* CLOCK_S(S, INPUT_BIT_S, CONTROL_BIT_S) -- spec [5]. */
static void clock_s(m2_state* st, int input_bit_s, int control_bit_s)
{
    uint8_t s_hat[M2_LEN], s_new[M2_LEN];
    int feedback_bit = st->s[99] ^ input_bit_s;
    int i;
    /* s^_0 = 0; s^_99 = s_98;
     * s^_i = s_{i-1} ^ ((s_i ^ COMP0_i) & (s_{i+1} ^ COMP1_i)), 1 <= i <= 98 */
    s_hat[0] = 0;
    for (i = 1; i <= 98; i++)
        s_hat[i] = (uint8_t)(st->s[i - 1] ^
                             ((st->s[i] ^ tbl(COMP0, i)) & (st->s[i + 1] ^ tbl(COMP1, i))));
    s_hat[99] = st->s[98];
    /* s'_i = s^_i ^ (FB0_i & FEEDBACK_BIT) if CONTROL_BIT_S == 0,
     *        s^_i ^ (FB1_i & FEEDBACK_BIT) otherwise */
    for (i = 0; i < M2_LEN; i++) {
        int fb = control_bit_s ? tbl(FB1, i) : tbl(FB0, i);
        s_new[i] = (uint8_t)(s_hat[i] ^ (fb & feedback_bit));
    }
    memcpy(st->s, s_new, M2_LEN);
}

/* CLOCK_KG(R, S, MIXING, INPUT_BIT) -- spec [5]; Fig. 2 / Fig. 9. */
static void clock_kg(m2_state* st, int mixing, int input_bit)
{
    int control_bit_r = st->s[34] ^ st->r[67];
    int control_bit_s = st->s[67] ^ st->r[33];
    int input_bit_r = mixing ? (input_bit ^ st->s[50]) : input_bit;
    int input_bit_s = input_bit;
    /* every bit that crosses between R and S (control and mixing bits) was
     * read above from the state before this call; CLOCK_R touches only R and
     * CLOCK_S only S, so running them in sequence is the spec's simultaneous
     * update */
    clock_r(st, input_bit_r, control_bit_r);
    clock_s(st, input_bit_s, control_bit_s);
}

/* Bit i of a byte string, MSB-first (spec [5] reference convention;
 * DESIGN.md reading R6). */
static int msb_bit(const uint8_t* buf, int i) { return (buf[i / 8] >> (7 - (i % 8))) & 1; }

/* Key/IV loading and preclock -- spec [5]:
 *   R = S = 0; for i < iv_bits: CLOCK_KG(1, iv_i); for i < 80: CLOCK_KG(1, k_i);
 *   100 x CLOCK_KG(1, 0). */
static void init(m2_state* st, const uint8_t key[10], const uint8_t* iv, int iv_bits)
{
    int i;
    memset(st, 0, sizeof(*st));
    for (i = 0; i < iv_bits; i++) clock_kg(st, 1, msb_bit(iv, i));
    for (i = 0; i < 80; i++) clock_kg(st, 1, msb_bit(key, i));
    for (i = 0; i < 100; i++) clock_kg(st, 1, 0);
}

/* ------------------------------- public API ------------------------------ */

/* Keystream of one instance: nbits bits, packed MSB-first into
 * out[0 .. ceil(nbits/8)), trailing bits of the last byte zero.
 * Keystream bit = r0 ^ s0, then CLOCK_KG(0, 0)  (spec [5]).
 * Returns 0, or -1 if iv_bits is outside [0, 80]. */
int ref_mickey2_keystream(const uint8_t key[10], const uint8_t* iv, int iv_bits,
                          uint64_t nbits, uint8_t* out)
{
    m2_state st;
    uint64_t t;
    if (iv_bits < 0 || iv_bits > 80) return -1;
    init(&st, key, iv, iv_bits);
    memset(out, 0, (size_t)((nbits + 7) / 8));
    for (t = 0; t < nbits; t++) {
        int z = st.r[0] ^ st.s[0];
        out[t / 8] |= (uint8_t)(z << (7 - (t % 8)));
        clock_kg(&st, 0, 0);
    }
    return 0;
}

/* State after init plus `extra_clocks` keystream clocks (preclock-parity hook):
 * r_out[i] = r_i, s_out[i] = s_i, one byte (0/1) per bit. */
int ref_mickey2_state(const uint8_t key[10], const uint8_t* iv, int iv_bits,
                      uint64_t extra_clocks, uint8_t* r_out, uint8_t* s_out)
{
    m2_state st;
    uint64_t t;
    if (iv_bits < 0 || iv_bits > 80) return -1;
    init(&st, key, iv, iv_bits);
    for (t = 0; t < extra_clocks; t++) clock_kg(&st, 0, 0);
    memcpy(r_out, st.r, M2_LEN);
    memcpy(s_out, st.s, M2_LEN);
    return 0;
}

/* One CLOCK_KG step on an explicit state (for algebraic pin tests).
 * r, s: 100 bytes each (0/1), updated in place. */
void ref_mickey2_clock_kg(uint8_t* r, uint8_t* s, int mixing, int input_bit)
{
    m2_state st;
    memcpy(st.r, r, M2_LEN);
    memcpy(st.s, s, M2_LEN);
    clock_kg(&st, mixing, input_bit);
    memcpy(r, st.r, M2_LEN);
    memcpy(s, st.s, M2_LEN);
}

/* Expose the spec table rows (for the table-invariant tests). which:
 * 0 = RTAPS membership, 1 = COMP0, 2 = COMP1, 3 = FB0, 4 = FB1.  Returns 0/1. */
int ref_mickey2_table(int which, int i)
{
    int t;
    if (i < 0 || i >= M2_LEN) return -1;
    switch (which) {
    case 0:
        for (t = 0; t < N_RTAPS; t++)
            if (RTAPS[t] == i) return 1;
        return 0;
    case 1: return tbl(COMP0, i);
    case 2: return tbl(COMP1, i);
    case 3: return tbl(FB0, i);
    case 4: return tbl(FB1, i);
    default: return -1;
    }
}
