/*
 * oracle/aes_ref.c -- byte-oriented AES-128 (FIPS-197) and CTR mode
 * (SP 800-38A) reference, CPU, plain C99.
 *
 * TEST INFRASTRUCTURE ONLY (see oracle/mickey2_ref.c for the rule).
 *
 * PAPER.md:288-307 (sec. 2.3.2): AES, a 4x4 byte state, 10 rounds for a
 * 128-bit key, SubBytes / ShiftRows / MixColumns / AddRoundKey; PAPER.md:
 * 307-338 (Fig. 3): AES in counter mode as a PRNG -- nonce||counter blocks,
 * the counter incremented per block, one 128-bit output block per counter
 * value; "different counter values ... with a unique key".
 * The cipher itself is FIPS-197 (ref [35]), written out
 * below in the standard's order: the S-box is COMPUTED from its definition
 * (multiplicative inverse in GF(2^8) mod x^8+x^4+x^3+x+1, then the affine map
 * with constant 0x63), not transcribed.  Reading A1: the counter
 * block is a 128-bit big-endian integer incremented by one per block
 * (SP 800-38A, Appendix B.1 standard incrementing function over all 128 bits).
 *
 * Pins (tests/test_oracle_aes.py): FIPS-197 C.1 and Appendix B, SP 800-38A
 * F.5.1 (golden fixture), and the `cryptography` library's AES-CTR.
 */
#include <stdint.h>
#include <string.h>

static uint8_t gf_mul(uint8_t a, uint8_t b)
{
    uint8_t r = 0;
    while (b) {
        if (b & 1) r ^= a;
        a = (uint8_t)((a << 1) ^ ((a & 0x80) ? 0x1b : 0x00));
        b >>= 1;
    }
    return r;
}

/* S-box (FIPS-197 sec. 5.1.1): b = x^-1 in GF(2^8) (0 -> 0), then
 * b'_i = b_i + b_{i+4} + b_{i+5} + b_{i+6} + b_{i+7} + c_i, c = 0x63. */
static uint8_t sbox_of(uint8_t x)
{
    uint8_t inv = 0, s = 0;
    int i, y;
    if (x)
        for (y = 1; y < 256; y++)
            if (gf_mul(x, (uint8_t)y) == 1) {
                inv = (uint8_t)y;
                break;
            }
    for (i = 0; i < 8; i++) {
        int bit = ((inv >> i) ^ (inv >> ((i + 4) % 8)) ^ (inv >> ((i + 5) % 8)) ^ (inv >> ((i + 6) % 8)) ^
                   (inv >> ((i + 7) % 8)) ^ (0x63 >> i)) & 1;
        s |= (uint8_t)(bit << i);
    }
    return s;
}

static uint8_t SBOX[256];
static int sbox_ready = 0;

static void init_sbox(void)
{
    int x;
    if (sbox_ready) return;
    for (x = 0; x < 256; x++) SBOX[x] = sbox_of((uint8_t)x);
    sbox_ready = 1;
}

/* KeyExpansion (FIPS-197 sec. 5.2), Nk = 4, Nr = 10: w[0..43] as bytes. */
static void key_expansion(const uint8_t key[16], uint8_t w[176])
{
    uint8_t rcon = 0x01;
    int i;
    memcpy(w, key, 16);
    for (i = 4; i < 44; i++) {
        uint8_t t[4];
        memcpy(t, w + 4 * (i - 1), 4);
        if (i % 4 == 0) {
            uint8_t t0 = t[0]; /* RotWord */
            t[0] = SBOX[t[1]];
            t[1] = SBOX[t[2]];
            t[2] = SBOX[t[3]];
            t[3] = SBOX[t0];
            t[0] ^= rcon; /* Rcon[i/Nk] = {rcon, 0, 0, 0} */
            rcon = gf_mul(rcon, 2);
        }
        w[4 * i + 0] = w[4 * (i - 4) + 0] ^ t[0];
        w[4 * i + 1] = w[4 * (i - 4) + 1] ^ t[1];
        w[4 * i + 2] = w[4 * (i - 4) + 2] ^ t[2];
        w[4 * i + 3] = w[4 * (i - 4) + 3] ^ t[3];
    }
}

/* state[r][c] = in[r + 4c] (FIPS-197 sec. 3.4) */
static void add_round_key(uint8_t s[4][4], const uint8_t* rk)
{
    int r, c;
    for (c = 0; c < 4; c++)
        for (r = 0; r < 4; r++) s[r][c] ^= rk[r + 4 * c];
}

static void sub_bytes(uint8_t s[4][4])
{
    int r, c;
    for (r = 0; r < 4; r++)
        for (c = 0; c < 4; c++) s[r][c] = SBOX[s[r][c]];
}

/* s'[r][c] = s[r][(c + r) mod 4] */
static void shift_rows(uint8_t s[4][4])
{
    uint8_t t[4][4];
    int r, c;
    for (r = 0; r < 4; r++)
        for (c = 0; c < 4; c++) t[r][c] = s[r][(c + r) % 4];
    memcpy(s, t, 16);
}

/* s'(x) = a(x) s(x) mod x^4+1, a(x) = {03}x^3 + {01}x^2 + {01}x + {02} */
static void mix_columns(uint8_t s[4][4])
{
    int c;
    for (c = 0; c < 4; c++) {
        uint8_t a0 = s[0][c], a1 = s[1][c], a2 = s[2][c], a3 = s[3][c];
        s[0][c] = gf_mul(a0, 2) ^ gf_mul(a1, 3) ^ a2 ^ a3;
        s[1][c] = a0 ^ gf_mul(a1, 2) ^ gf_mul(a2, 3) ^ a3;
        s[2][c] = a0 ^ a1 ^ gf_mul(a2, 2) ^ gf_mul(a3, 3);
        s[3][c] = gf_mul(a0, 3) ^ a1 ^ a2 ^ gf_mul(a3, 2);
    }
}

/* Cipher (FIPS-197 sec. 5.1) with an expanded key. */
static void cipher(const uint8_t w[176], const uint8_t in[16], uint8_t out[16])
{
    uint8_t s[4][4];
    int r, c, round;
    for (c = 0; c < 4; c++)
        for (r = 0; r < 4; r++) s[r][c] = in[r + 4 * c];
    add_round_key(s, w);
    for (round = 1; round < 10; round++) {
        sub_bytes(s);
        shift_rows(s);
        mix_columns(s);
        add_round_key(s, w + 16 * round);
    }
    sub_bytes(s);
    shift_rows(s);
    add_round_key(s, w + 160);
    for (c = 0; c < 4; c++)
        for (r = 0; r < 4; r++) out[r + 4 * c] = s[r][c];
}

/* ------------------------------- public API ------------------------------ */

void ref_aes128_encrypt_block(const uint8_t key[16], const uint8_t in[16], uint8_t out[16])
{
    uint8_t w[176];
    init_sbox();
    key_expansion(key, w);
    cipher(w, in, out);
}

void ref_aes128_expand_key(const uint8_t key[16], uint8_t w[176])
{
    init_sbox();
    key_expansion(key, w);
}

uint8_t ref_aes_sbox(uint8_t x)
{
    init_sbox();
    return SBOX[x];
}

/* CTR keystream (SP 800-38A sec. 6.5): blocks E_K(T_j), T_{j+1} = T_j + 1 mod
 * 2^128 (big-endian).  Starting at block index `first_block` (i.e. T = ctr +
 * first_block), nblocks blocks are written to out (16 bytes each). */
void ref_aes128_ctr_keystream(const uint8_t key[16], const uint8_t ctr[16], uint64_t first_block,
                              uint64_t nblocks, uint8_t* out)
{
    uint8_t w[176], t[16];
    uint64_t j;
    int k;
    init_sbox();
    key_expansion(key, w);
    memcpy(t, ctr, 16);
    /* t += first_block (128-bit big-endian add) */
    {
        uint64_t add = first_block;
        unsigned carry = 0;
        for (k = 15; k >= 0; k--) {
            unsigned v = t[k] + (unsigned)(add & 0xff) + carry;
            t[k] = (uint8_t)v;
            carry = v >> 8;
            add >>= 8;
        }
    }
    for (j = 0; j < nblocks; j++) {
        cipher(w, t, out + 16 * j);
        for (k = 15; k >= 0; k--) /* increment */
            if (++t[k] != 0) break;
    }
}
