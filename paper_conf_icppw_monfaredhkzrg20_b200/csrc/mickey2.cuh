// mickey2.cuh -- bitsliced MICKEY 2.0 for sm_100a.
//
// PAPER.md:597-656 (sec. 4.4, Fig. 9): "instead of two 100-bit registers ...
// 200 registers, each containing 32 bits are employed ... each GPU thread can
// execute 32 parallel Mickey 2.0 ciphers, and each thread at each clock cycle
// generates 32 random bits."  The per-bit procedures are those of the MICKEY
// 2.0 specification (ref [5]); here every bit r_i / s_i is a
// 32-lane slice word and every step is one 3-input logic op (LOP3).
//
// The tables below are the GPU-side encoding (packed masks, bit i at word
// i/32, bit i%32).  They are NOT shared with the oracle, which transcribes the
// specification's bit rows; tests/test_oracle_mickey2.py checks the two
// encodings agree.
//
// Op count per keystream clock: R 149, S 174, fb0/fb1 2,
// control 1, output 1 = 327 LOP3 for 32 keystream bits.
#pragma once
#include <cstdint>
#include <utility>

#include "bitslice.cuh"

namespace bsk {
namespace m2 {

__host__ __device__ constexpr uint32_t pick(uint32_t w0, uint32_t w1, uint32_t w2, uint32_t w3, int i)
{
    return ((i < 32 ? w0 : i < 64 ? w1 : i < 96 ? w2 : w3) >> (i & 31)) & 1u;
}
// RTAPS (50 taps), COMP0/COMP1 (used for 1 <= i <= 98), FB0, FB1.
__host__ __device__ constexpr bool rtap(int i) { return pick(0x1279327Bu, 0xB5546660u, 0xDF87818Fu, 0x00000003u, i); }
__host__ __device__ constexpr uint32_t comp0(int i) { return pick(0x6AA97A30u, 0x7942A809u, 0x057EBFEAu, 0x00000006u, i) ? 0xFFFFFFFFu : 0u; }
__host__ __device__ constexpr uint32_t comp1(int i) { return pick(0xDD629E9Au, 0xE3A21D63u, 0x91C23DD7u, 0x00000001u, i) ? 0xFFFFFFFFu : 0u; }
__host__ __device__ constexpr bool fb0(int i) { return pick(0x9FFA7FAFu, 0xAF4A9381u, 0x9CEC5802u, 0x00000001u, i); }
__host__ __device__ constexpr bool fb1(int i) { return pick(0x4C8CB877u, 0x4911B063u, 0x40FBC52Bu, 0x00000008u, i); }

constexpr int NSTATE = 200;

// a ^ (b & c) as one explicit LOP3 (bsk::lop3, bitslice.cuh).  Given the C
// expression, the compiler folds CONTROL_BIT_R = s34 ^ r67 into every AND
// (r_i & (s34 ^ r67) is one 3-input LOP3) and then needs a second LOP3 for the
// XOR with r_{i-1}: 2 ops per bit instead of 1 (+50 ops per clock).
constexpr uint32_t LUT_A_XOR_BC = 0xF0u ^ (0xCCu & 0xAAu);  // 0x78

template <int I>
__device__ __forceinline__ uint32_t s_next(const uint32_t (&s)[100], uint32_t fb_s, uint32_t fb_s0, uint32_t fb_s1)
{
    uint32_t v;
    if constexpr (I == 0) {
        v = 0u;
    } else if constexpr (I == 99) {
        v = s[98];
    } else {
        constexpr uint32_t c0 = comp0(I) & 0xFFu, c1 = comp1(I) & 0xFFu;
        constexpr uint32_t LUT = 0xF0u ^ ((0xCCu ^ c0) & (0xAAu ^ c1));
        v = lop3<LUT>(s[I - 1], s[I], s[I + 1]);
    }
    if constexpr (fb0(I) && fb1(I))
        v = (I == 0) ? fb_s : (v ^ fb_s);
    else if constexpr (fb0(I))
        v ^= fb_s0;
    else if constexpr (fb1(I))
        v ^= fb_s1;
    return v;
}

template <int... I>
__device__ __forceinline__ void s_update(uint32_t (&ns)[100], const uint32_t (&s)[100], uint32_t fb_s, uint32_t fb_s0,
                                         uint32_t fb_s1, std::integer_sequence<int, I...>)
{
    ((ns[I] = s_next<I>(s, fb_s, fb_s0, fb_s1)), ...);
}

// One CLOCK_KG on 32 lanes.  MIX = the spec's MIXING flag (init clocks);
// `in` = INPUT_BIT slice word (ignored unless MIX).
//   CONTROL_BIT_R = s34 ^ r67, CONTROL_BIT_S = s67 ^ r33   (Fig. 2)
//   FEEDBACK_R = r99 ^ in ^ (MIX ? s50 : 0), FEEDBACK_S = s99 ^ in
//   r'_i = r_{i-1} ^ [i in RTAPS] fbR ^ (ctlR & r_i)          (r_{-1} = 0)
//   s'_i = s^_i ^ (FB0_i & fbS & ~ctlS) ^ (FB1_i & fbS & ctlS)
//   s^_i = s_{i-1} ^ ((s_i ^ COMP0_i) & (s_{i+1} ^ COMP1_i)), s^_0 = 0, s^_99 = s_98
// R is updated in place top-down (old r_i is read only by r'_i and r'_{i+1});
// S goes through a renamed array (every old s_i is read by three updates), which
// after full unrolling is pure register renaming.
template <bool MIX, int NR>
__device__ __forceinline__ void clock_kg(uint32_t (&r)[NR], uint32_t (&s)[100], uint32_t in)
{
    const uint32_t ctl_r = s[34] ^ r[67];
    const uint32_t ctl_s = s[67] ^ r[33];
    const uint32_t fb_r = MIX ? (r[99] ^ in ^ s[50]) : r[99];
    const uint32_t fb_s = MIX ? (s[99] ^ in) : s[99];
    const uint32_t fb_s0 = fb_s & ~ctl_s;  // FB0 taps apply where CONTROL_BIT_S = 0
    const uint32_t fb_s1 = fb_s & ctl_s;   // FB1 taps apply where CONTROL_BIT_S = 1

#pragma unroll
    for (int i = 99; i >= 1; --i) {
        const uint32_t a = rtap(i) ? (r[i - 1] ^ fb_r) : r[i - 1];
        r[i] = lop3<LUT_A_XOR_BC>(a, ctl_r, r[i]);
    }
    r[0] = lop3<LUT_A_XOR_BC>(fb_r, ctl_r, r[0]);  // 0 is in RTAPS

    uint32_t ns[100];
    s_update(ns, s, fb_s, fb_s0, fb_s1, std::make_integer_sequence<int, 100>{});
#pragma unroll
    for (int i = 0; i < 100; ++i) s[i] = ns[i];
}

// ---------------------------------------------------------------------------
// Keystream clocks with the Galois reduction of R deferred over a block of K
// clocks (K = 2, 4 or 8; B200 design, not the paper's).
//
// In polynomial form (spec [5]: r'_i = r_{i-1} ^ [i in RTAPS] r99 ^ (ctlR & r_i))
// the R clock is R' = (x + ctlR) * R mod p(x), p(x) = x^100 + sum_{t in RTAPS}
// x^t, lane by lane.  Multiplication commutes with the reduction, so within a
// block we keep an unreduced P == R (mod p) whose degree grows by one per
// clock: P' = (x + ctlR) * P costs one LOP3 per position and no feedback taps
// (the new top word is a rename).  At the block's end the K overflow words
// h_m = P_{100+m} are folded back, h_m * x^(100+m) mod p = h_m * Q_m(x): each
// low position q receives the XOR of the h_m with q in Q_m.  Pairs of h words
// are pre-combined (h_0^h_1, h_2^h_3, ...), so a position takes at most one
// operand per pair: one LOP3 per position at K = 4 instead of one per tap per
// clock.  The three taps the clock reads mid-block (r0 for z, r33 for
// CONTROL_BIT_S, r67 for CONTROL_BIT_R) add their pending h_m terms explicitly.
//
// Ops per clock for R at K = 4: 101.5 (shift) + 1.25 (tap corrections) + 23.25
// (reduction incl. 2 pair combos) = 126 vs 149 in Galois form, so a keystream
// clock is 304 LOP3 instead of 327 (`lazy_ops_per_clock`).
// Bit-exactness: at every block boundary P is fully reduced and equals the
// spec's R (the state carry and the parity tests see only reduced states).
// ---------------------------------------------------------------------------
constexpr int KMAX = 8;  // largest block; Q_0..Q_7

struct QTab {
    uint32_t w[KMAX][4];
};
// Q_m = x^(100+m) mod p(x) as bit masks (bit q of word q/32)
__host__ __device__ constexpr QTab make_qtab()
{
    QTab t{};
    uint32_t cur[4] = {0x1279327Bu, 0xB5546660u, 0xDF87818Fu, 0x00000003u};  // x^100 = sum RTAPS x^t
    for (int m = 0; m < KMAX; ++m) {
        for (int i = 0; i < 4; ++i) t.w[m][i] = cur[i];
        const uint32_t carry = (cur[3] >> 3) & 1u;  // bit 99
        cur[3] = ((cur[3] << 1) | (cur[2] >> 31)) & 0xFu;
        cur[2] = (cur[2] << 1) | (cur[1] >> 31);
        cur[1] = (cur[1] << 1) | (cur[0] >> 31);
        cur[0] = cur[0] << 1;
        if (carry) {
            cur[0] ^= 0x1279327Bu;
            cur[1] ^= 0xB5546660u;
            cur[2] ^= 0xDF87818Fu;
            cur[3] ^= 0x00000003u;
        }
    }
    return t;
}
__host__ __device__ constexpr bool qbit(int m, int q)
{
    return (make_qtab().w[m][q >> 5] >> (q & 31)) & 1u;
}
// pending words m < J that feed position q, and the i-th of them
__host__ __device__ constexpr int n_terms(int q, int J)
{
    int n = 0;
    for (int m = 0; m < J; ++m) n += qbit(m, q) ? 1 : 0;
    return n;
}
__host__ __device__ constexpr int term_m(int q, int J, int i)
{
    for (int m = 0; m < J; ++m)
        if (qbit(m, q) && i-- == 0) return m;
    return -1;
}

constexpr int RN = 100 + KMAX;  // R register words incl. pending positions
constexpr uint32_t XOR2 = 0x3Cu, XOR3 = 0x96u, AND2 = 0xC0u;

// XOR of: e[0..NE-1], r[Q] and the pending terms of position Q at phase J
// (the true spec bit r_Q mid-block), two operands per LOP3.
template <int Q, int J, int NE, int K>
__device__ __forceinline__ uint32_t opnd(const uint32_t (&e)[NE], const uint32_t (&r)[RN])
{
    if constexpr (K < NE)
        return e[K];
    else if constexpr (K == NE)
        return r[Q];
    else
        return r[100 + term_m(Q, J, K - NE - 1)];
}
template <int Q, int J, int NE, int K, int NT>
__device__ __forceinline__ uint32_t fold(uint32_t v, const uint32_t (&e)[NE], const uint32_t (&r)[RN])
{
    if constexpr (K + 1 < NT)
        return fold<Q, J, NE, K + 2, NT>(lop3<XOR3>(v, opnd<Q, J, NE, K>(e, r), opnd<Q, J, NE, K + 1>(e, r)), e, r);
    else if constexpr (K < NT)
        return lop3<XOR2>(v, opnd<Q, J, NE, K>(e, r), 0u);
    else
        return v;
}
template <int Q, int J, int NE>
__device__ __forceinline__ uint32_t xor_true(const uint32_t (&e)[NE], const uint32_t (&r)[RN])
{
    constexpr int NT = NE + 1 + n_terms(Q, J);
    return fold<Q, J, NE, 1, NT>(opnd<Q, J, NE, 0>(e, r), e, r);
}

// End-of-block reduction: r[q] ^= sum_{m < K, q in Q_m} h_m, h_m = r[100+m].
// Operand of pair p for position q: h_{2p}, h_{2p+1} or their pre-combined XOR.
template <int K>
__device__ __forceinline__ uint32_t pair_opnd(const uint32_t (&r)[RN], const uint32_t (&cmb)[KMAX / 2], int p, int q)
{
    const bool a = qbit(2 * p, q), b = K > 2 * p + 1 && qbit(2 * p + 1, q);
    return a && b ? cmb[p] : a ? r[100 + 2 * p] : r[101 + 2 * p];
}
__host__ __device__ constexpr bool pair_used(int K, int p, int q)
{
    return qbit(2 * p, q) || (K > 2 * p + 1 && qbit(2 * p + 1, q));
}
__host__ __device__ constexpr int n_pairs_used(int K, int q)
{
    int n = 0;
    for (int p = 0; p < (K + 1) / 2; ++p) n += pair_used(K, p, q) ? 1 : 0;
    return n;
}
__host__ __device__ constexpr int pair_i(int K, int q, int i)
{
    for (int p = 0; p < (K + 1) / 2; ++p)
        if (pair_used(K, p, q) && i-- == 0) return p;
    return -1;
}
__host__ __device__ constexpr bool combo_needed(int K, int p)
{
    if (K <= 2 * p + 1) return false;
    for (int q = 0; q < 100; ++q)
        if (qbit(2 * p, q) && qbit(2 * p + 1, q)) return true;
    return false;
}
template <int K, int Q, int I, int N>
__device__ __forceinline__ uint32_t red_fold(uint32_t v, const uint32_t (&r)[RN], const uint32_t (&cmb)[KMAX / 2])
{
    if constexpr (I + 1 < N)
        return red_fold<K, Q, I + 2, N>(
            lop3<XOR3>(v, pair_opnd<K>(r, cmb, pair_i(K, Q, I), Q), pair_opnd<K>(r, cmb, pair_i(K, Q, I + 1), Q)), r,
            cmb);
    else if constexpr (I < N)
        return lop3<XOR2>(v, pair_opnd<K>(r, cmb, pair_i(K, Q, I), Q), 0u);
    else
        return v;
}
template <int K, int... Q>
__device__ __forceinline__ void reduce(uint32_t (&r)[RN], std::integer_sequence<int, Q...>)
{
    uint32_t cmb[KMAX / 2];
#pragma unroll
    for (int p = 0; p < KMAX / 2; ++p) cmb[p] = 0u;
    if constexpr (combo_needed(K, 0)) cmb[0] = lop3<XOR2>(r[100], r[101], 0u);
    if constexpr (combo_needed(K, 1)) cmb[1] = lop3<XOR2>(r[102], r[103], 0u);
    if constexpr (combo_needed(K, 2)) cmb[2] = lop3<XOR2>(r[104], r[105], 0u);
    if constexpr (combo_needed(K, 3)) cmb[3] = lop3<XOR2>(r[106], r[107], 0u);
    ((r[Q] = red_fold<K, Q, 0, n_pairs_used(K, Q)>(r[Q], r, cmb)), ...);
}

// The S half of CLOCK_KG, given CONTROL_BIT_S and FEEDBACK_S.
__device__ __forceinline__ void s_clock(uint32_t (&s)[100], uint32_t ctl_s, uint32_t fb_s)
{
    const uint32_t fb_s0 = fb_s & ~ctl_s;
    const uint32_t fb_s1 = fb_s & ctl_s;
    uint32_t ns[100];
    s_update(ns, s, fb_s, fb_s0, fb_s1, std::make_integer_sequence<int, 100>{});
#pragma unroll
    for (int i = 0; i < 100; ++i) s[i] = ns[i];
}

// Clock J (0..K-1) of a K-clock block.  Before it, r[100..99+J] hold the
// pending overflow words; after clock K-1, R is reduced again.  MIX = the
// spec's MIXING (initialisation): FEEDBACK_R gains u = INPUT_BIT ^ s50, i.e.
// R' = (x + c) R + u * sum_{t in RTAPS} x^t = (x + c) R + u * x^100 (mod p), so
// u is XORed into the pending word at position 100 (one op, not one per tap);
// FEEDBACK_S = s99 ^ INPUT_BIT.
template <int J, int K, bool MIX = false>
__device__ __forceinline__ void clock_lazy(uint32_t (&r)[RN], uint32_t (&s)[100], uint32_t in = 0u)
{
    static_assert(K >= 2 && K <= KMAX && J < K, "block of 2..8 clocks");
    const uint32_t e34[1] = {s[34]}, e67[1] = {s[67]};
    const uint32_t ctl_r = xor_true<67, J, 1>(e34, r);  // s34 ^ r67
    const uint32_t ctl_s = xor_true<33, J, 1>(e67, r);  // s67 ^ r33
    const uint32_t u = MIX ? lop3<XOR2>(in, s[50], 0u) : 0u;
    const uint32_t fb_s = MIX ? lop3<XOR2>(s[99], in, 0u) : s[99];
    if constexpr (MIX && J == 0)
        r[100] = lop3<XOR2>(r[99], u, 0u);  // top word: rename, + u x^100
    else
        r[100 + J] = r[99 + J];             // top word: rename
#pragma unroll
    for (int i = 99 + J; i >= 1; --i) {
        if (MIX && J > 0 && i == 100)
            r[i] = lop3<XOR2>(lop3<LUT_A_XOR_BC>(r[i - 1], ctl_r, r[i]), u, 0u);
        else
            r[i] = lop3<LUT_A_XOR_BC>(r[i - 1], ctl_r, r[i]);
    }
    r[0] = lop3<AND2>(ctl_r, r[0], 0u);
    s_clock(s, ctl_s, fb_s);
    if constexpr (J == K - 1) reduce<K>(r, std::make_integer_sequence<int, 100>{});
}
// four initialisation clocks (MIXING = 1) with input words in[0..3]
__device__ __forceinline__ void clock4_mix(uint32_t (&r)[RN], uint32_t (&s)[100], const uint32_t (&in)[4])
{
    clock_lazy<0, 4, true>(r, s, in[0]);
    clock_lazy<1, 4, true>(r, s, in[1]);
    clock_lazy<2, 4, true>(r, s, in[2]);
    clock_lazy<3, 4, true>(r, s, in[3]);
}

}  // namespace m2
}  // namespace bsk

namespace bsk {

// Cipher traits used by keystream_kernel (keystream.cuh).
struct Mickey2 {
    static constexpr int NSTATE = m2::NSTATE;
    static constexpr bool MSB_FIRST = true;  // spec [5]: keystream packed MSB-first
    // clocks per loop iteration: 4 keeps the loop (21 KB of SASS) in the
    // instruction cache.  Only U = 4 is built: U = 8 overflowed the cache
    // (0.92 of roofline, 270 B of stack) and at U = 2 ptxas put the whole
    // consume state in local memory (round-1 sweep).
    static constexpr int U_DEFAULT = 4, U_ALT0 = 4, U_ALT1 = 4;
    // ROW_MAJOR default: the plain clock kernel with row segments staged in
    // TMEM, two CTAs per SM, one work item per warp-unit (0.935 of the ALU
    // roofline vs 0.904 for the smem warp-specialised kernel)
    static constexpr bool RM_TMEM = true, RM_SEGMENTED = false;
    // ROW_MAJOR warp-specialised kernel (rowmajor_ws.cuh) only when every
    // warp-unit gets its own SMSP (the paper shape: C4 1.41 vs 1.37 Tb/s);
    // otherwise two clock-loop warps per SMSP keep the ALU fuller than one
    // plus a writer (C2 1.85 vs 1.81)
    static constexpr int RM_WS = 1;
    // r[100..107]: pending overflow words of the deferred R reduction
    // (clock_at); only positions 0..99 are state between blocks
    uint32_t r[m2::RN], s[100];
    // clocks per deferred-reduction block for a U-clock loop body
    static constexpr int block_k(int U) { return U % 4 == 0 ? 4 : U % 2 == 0 ? 2 : 1; }

    // State carry (SURVEY step a-5).  The row pointer goes through opaque()
    // so the 200 load addresses are not kept live across the clock loop for
    // reuse by the stores (that would cost 400 registers).
    __device__ __forceinline__ void load(const uint32_t* st, uint64_t Gp, uint64_t g)
    {
        const uint32_t* p = opaque(st + g);
#pragma unroll
        for (int i = 0; i < 100; ++i) r[i] = __ldcg(p + uint64_t(i) * Gp);
#pragma unroll
        for (int i = 0; i < 100; ++i) s[i] = __ldcg(p + uint64_t(100 + i) * Gp);
    }
    __device__ __forceinline__ void store(uint32_t* st, uint64_t Gp, uint64_t g) const
    {
        uint32_t* p = opaque(st + g);
#pragma unroll
        for (int i = 0; i < 100; ++i) __stcg(p + uint64_t(i) * Gp, r[i]);
#pragma unroll
        for (int i = 0; i < 100; ++i) __stcg(p + uint64_t(100 + i) * Gp, s[i]);
    }
    // keystream bit z = r0 ^ s0, taken before the clock (spec [5])
    __device__ __forceinline__ uint32_t z() const { return r[0] ^ s[0]; }
    __device__ __forceinline__ uint32_t z_acc(uint32_t acc) const { return acc ^ r[0] ^ s[0]; }
    __device__ __forceinline__ void clock() { m2::clock_kg<false>(r, s, 0u); }
    // clock J of a K-clock deferred-reduction block (K = block_k(U) > 1)
    template <int J, int K>
    __device__ __forceinline__ uint32_t z_at() const
    {
        const uint32_t e[1] = {s[0]};
        return m2::xor_true<0, J, 1>(e, r);
    }
    template <int J, int K>
    __device__ __forceinline__ uint32_t z_acc_at(uint32_t acc) const
    {
        const uint32_t e[2] = {acc, s[0]};
        return m2::xor_true<0, J, 2>(e, r);
    }
    template <int J, int K>
    __device__ __forceinline__ void clock_at()
    {
        m2::clock_lazy<J, K>(r, s);
    }
};

// Initialisation (SURVEY step a-2, spec [5]): R = S = 0,
// then CLOCK_KG(MIXING=1, INPUT_BIT) for the iv_bits IV bits, the 80 key bits
// and 100 zero bits.  One thread per group; one coalesced slice word per clock.
//   iv_s, key_s: uint32 [80][Gp] sliced bits (slice_bits_kernel)
//   state      : uint32 [201][Gp] (row 200 = checksum accumulator, zeroed)
__global__ void __launch_bounds__(128) m2_preclock_kernel(const uint32_t* __restrict__ iv_s,
                                                          const uint32_t* __restrict__ key_s,
                                                          int iv_bits, uint32_t* __restrict__ state,
                                                          uint64_t Gp)
{
    const uint64_t g = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (g >= Gp) return;
    uint32_t r[100], s[100];
#pragma unroll
    for (int i = 0; i < 100; ++i) r[i] = s[i] = 0u;
    // The spec's input sequence is iv_bits IV bits, 80 key bits, then 100
    // zero bits: T = iv_bits + 180 mixing clocks, 4 per loop iteration (the
    // S-register renaming closes inside the body), then the last T mod 4
    // (< 100, so zero-input) clocks one at a time -- any iv_bits in 0..80.
    const int nin = iv_bits + 80, T = nin + 100, T4 = T & ~3;
    const uint32_t* iv_p = iv_s + g;
    const uint32_t* key_p = key_s + g - uint64_t(iv_bits) * Gp;
    auto in_word = [&](int c) { return c < nin ? __ldcs((c < iv_bits ? iv_p : key_p) + uint64_t(c) * Gp) : 0u; };
#pragma unroll 1
    for (int c = 0; c < T4; c += 4) {
        uint32_t in[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) in[u] = in_word(c + u);
#pragma unroll
        for (int u = 0; u < 4; ++u) m2::clock_kg<true>(r, s, in[u]);
    }
#pragma unroll 1
    for (int c = T4; c < T; ++c) m2::clock_kg<true>(r, s, 0u);
#pragma unroll
    for (int i = 0; i < 100; ++i) state[uint64_t(i) * Gp + g] = r[i];
#pragma unroll
    for (int i = 0; i < 100; ++i) state[uint64_t(100 + i) * Gp + g] = s[i];
    state[uint64_t(200) * Gp + g] = 0u;
}

}  // namespace bsk

namespace bsk {

// ---------------------------------------------------------------------------
// Fused key/IV slicing + preclock (SURVEY steps a-1 + a-2 in one kernel).
//
// The separate path (slice_bits_kernel x2 -> sliced words in HBM ->
// m2_preclock_kernel) spent ~20% of a rekey in the two slicing launches and
// re-read every input word from HBM inside the clock loop.  Here each thread
// (one group, as in the clock loop) loads its 32 instances' IV and key bytes
// with 16 B loads, slices them in registers (slice_group32: PRMT + the 32x32
// bit transpose) while the cipher state is still all-zero (no extra register
// pressure), and parks the 160 slice words in shared memory [bit][thread];
// the 260 mixing clocks then read their input word from shared memory.
// 20 KB of smem per warp -> two 4-warp CTAs (two warps per SMSP) per SM.
// Inputs: group g's 32 keys / IVs (10 B each) at raw_k / raw_iv + 320 g for
// g < g_split (16 B aligned; the caller's device arrays or the staging copy),
// else at tail_k / tail_iv + 320 (g - g_split) (zero beyond instance n).
// ---------------------------------------------------------------------------
constexpr int M2I_BLOCK = 128;
constexpr size_t M2I_SMEM_BYTES = size_t(160) * M2I_BLOCK * 4;  // [IV bit 0..79, key bit 0..79][thread]

__global__ void __launch_bounds__(M2I_BLOCK, 2) m2_init_kernel(const uint8_t* __restrict__ raw_k,
                                                              const uint8_t* __restrict__ raw_iv,
                                                              const uint8_t* __restrict__ tail_k,
                                                              const uint8_t* __restrict__ tail_iv, uint64_t g_split,
                                                              int iv_bits, uint32_t* __restrict__ state, uint64_t Gp)
{
    extern __shared__ uint32_t m2i_smem[];
    const uint64_t g = uint64_t(blockIdx.x) * M2I_BLOCK + threadIdx.x;
    if (g >= Gp) return;  // no block-level barrier below
    uint32_t* sl = m2i_smem + threadIdx.x;
    slice_group32<10, 80, true>(group_src(raw_iv, tail_iv, g_split, g, 320u),
                                [&](int bit, uint32_t w) { sl[bit * M2I_BLOCK] = w; });
    slice_group32<10, 80, true>(group_src(raw_k, tail_k, g_split, g, 320u),
                                [&](int bit, uint32_t w) { sl[(80 + bit) * M2I_BLOCK] = w; });

    // R with the deferred reduction (m2::clock_lazy, 4-clock blocks; reduced
    // again at every block boundary, so the stored state is the spec's)
    uint32_t r[m2::RN], s[100];
#pragma unroll
    for (int i = 0; i < 100; ++i) r[i] = s[i] = 0u;
    // T = iv_bits + 180 mixing clocks: IV bits (rows 0..iv_bits-1), key bits
    // (rows 80..159), 100 zero bits; 4-clock deferred-reduction blocks, then
    // the last T mod 4 (zero-input) clocks in Galois form, so any iv_bits in
    // 0..80 works (the block loop needs whole 4-clock blocks)
    const int nin = iv_bits + 80, T = nin + 100, T4 = T & ~3;
#pragma unroll 1
    for (int c = 0; c < T4; c += 4) {
        uint32_t in[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            const int cu = c + u;
            const int row = cu < iv_bits ? cu : cu - iv_bits + 80;
            in[u] = cu < nin ? sl[row * M2I_BLOCK] : 0u;
        }
        m2::clock4_mix(r, s, in);
    }
#pragma unroll 1
    for (int c = T4; c < T; ++c) m2::clock_kg<true>(r, s, 0u);
    uint32_t* p = opaque(state + g);
#pragma unroll
    for (int i = 0; i < 100; ++i) __stcg(p + uint64_t(i) * Gp, r[i]);
#pragma unroll
    for (int i = 0; i < 100; ++i) __stcg(p + uint64_t(100 + i) * Gp, s[i]);
    p[uint64_t(200) * Gp] = 0u;
}

}  // namespace bsk
