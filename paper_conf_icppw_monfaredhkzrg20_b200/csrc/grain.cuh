// grain.cuh -- bitsliced Grain v1 for sm_100a.
//
// PAPER.md:339-357 (sec. 2.3.3, Fig. 4): Grain, an 80-bit LFSR s and an 80-bit
// NFSR b, LFSR feedback f, NFSR feedback g, filter h; 80-bit key, 64-bit IV,
// 160 initialisation clocks; PAPER.md:456-460 and Fig. 10: the paper's second
// bitsliced stream cipher.  Definitions follow the Grain v1 specification
// (ref [15]).  One thread = 32 instances; every register bit
// is a 32-lane slice word.
//
// Both registers shift by one position per clock (Fibonacci form), so the
// shift is pure register renaming; only the three new words (f, g, z) cost
// logic: 37 LOP3 per clock per 32 keystream bits (f 3, g 25, h + z 9; SURVEY
// App. D estimated 39), ~9x cheaper than MICKEY 2.0.  The renaming closes every 80 clocks; with U clocks per loop
// iteration ptxas restores the register map at the back edge with moves
// (160/U per clock, issued on the otherwise idle FMA pipe).
#pragma once
#include <cstdint>

#include "bitslice.cuh"

namespace bsk {
namespace grain {

constexpr int NSTATE = 160;  // s_0..s_79, b_0..b_79

// LOP3 truth tables (a = 0xF0, b = 0xCC, c = 0xAA)
constexpr uint32_t XOR3 = 0x96u, XOR2 = 0x3Cu, AND3 = 0x80u, AND2 = 0xC0u;
constexpr uint32_t XAND = 0x78u;  // a ^ (b & c)
constexpr uint32_t MUX = 0xCAu;   // a ? b : c

// Output z = b1+b2+b4+b10+b31+b43+b56 + h(s3, s25, s46, s64, b63), with
//   h = x1 + x4 + x0x3 + x2x3 + x3x4 + x0x1x2 + x0x2x3 + x0x2x4 + x1x2x4 + x2x3x4
//     = x1 + (x3 ? x0 : x4) + x2 * B,
//   B = x0 ? (x1|x4) + x3x4 : x3 + x1x4 + x3x4          (x0 = s3, x1 = s25,
// x2 = s46, x3 = s64, x4 = b63; verified exhaustively in DESIGN.md's note).
// `extra` is XORed in (the checksum accumulator, or 0): 9 LOP3 (+1 with extra).
template <bool EXTRA>
__device__ __forceinline__ uint32_t output(const uint32_t (&s)[80], const uint32_t (&b)[80], uint32_t extra = 0u)
{
    const uint32_t x0 = s[3], x1 = s[25], x2 = s[46], x3 = s[64], x4 = b[63];
    const uint32_t m = lop3<MUX>(x3, x0, x4);
    const uint32_t B0 = lop3<0xE4u>(x1, x3, x4);  // x3 ^ x1x4 ^ x3x4
    const uint32_t B1 = lop3<0x72u>(x1, x3, x4);  // (x1 | x4) ^ x3x4
    const uint32_t B = lop3<MUX>(x0, B1, B0);
    const uint32_t w1 = lop3<XOR3>(b[1], b[2], b[4]);
    const uint32_t w2 = lop3<XOR3>(b[10], b[31], b[43]);
    const uint32_t w3 = lop3<XOR3>(b[56], x1, m);
    uint32_t w = lop3<XOR3>(w1, w2, w3);
    if (EXTRA) w = lop3<XOR2>(w, extra, 0u);
    return lop3<XAND>(w, x2, B);
}

// f: s_80 = s62+s51+s38+s23+s13+s0  (3 LOP3)
__device__ __forceinline__ uint32_t f_lfsr(const uint32_t (&s)[80])
{
    return lop3<XOR3>(lop3<XOR3>(s[62], s[51], s[38]), lop3<XOR3>(s[23], s[13], s[0]), 0u);
}

// g: b_80 = s0 + b62+b60+b52+b45+b37+b33+b28+b21+b14+b9+b0 + b63b60 + b37b33 + b15b9
//         + b60b52b45 + b33b28b21 + b63b45b28b9 + b60b52b37b33 + b63b60b21b15
//         + b63b60b52b45b37 + b33b28b21b15b9 + b52b45b37b33b28b21
// as a balanced LOP3 tree: 25 ops, depth 5 (the linear terms are grouped
// with single AND-products into a ^ (b & c) gates).
__device__ __forceinline__ uint32_t g_nfsr(uint32_t s0, const uint32_t (&b)[80])
{
    const uint32_t t1 = lop3<XOR3>(s0, b[62], b[60]);
    const uint32_t t2 = lop3<XOR3>(b[52], b[45], b[37]);
    const uint32_t t3 = lop3<XOR3>(b[33], b[28], b[21]);
    const uint32_t t4 = lop3<XOR3>(b[14], b[9], b[0]);
    const uint32_t q45 = lop3<AND2>(b[52], b[45], 0u);
    const uint32_t q21 = lop3<AND2>(b[28], b[21], 0u);
    const uint32_t p1 = lop3<AND2>(b[63], b[60], 0u);
    const uint32_t p2 = lop3<AND2>(b[37], b[33], 0u);
    const uint32_t p3 = lop3<AND2>(b[15], b[9], 0u);
    const uint32_t a1 = lop3<XAND>(t2, b[60], q45);        // + b60b52b45
    const uint32_t p5 = lop3<AND2>(b[33], q21, 0u);        // b33b28b21
    const uint32_t m1 = lop3<AND2>(b[63], b[45], 0u);
    const uint32_t m2 = lop3<AND2>(b[28], b[9], 0u);
    const uint32_t a2 = lop3<XAND>(t3, m1, m2);            // + b63b45b28b9
    const uint32_t p7 = lop3<AND3>(b[60], b[52], p2);      // b60b52b37b33
    const uint32_t p8 = lop3<AND3>(p1, b[21], b[15]);      // b63b60b21b15
    const uint32_t p9 = lop3<AND3>(p1, q45, b[37]);        // b63b60b52b45b37
    const uint32_t a3 = lop3<XAND>(t4, p5, p3);            // + b33b28b21b15b9
    const uint32_t p11 = lop3<AND3>(q45, p2, q21);         // b52b45b37b33b28b21
    const uint32_t u1 = lop3<XOR3>(t1, a1, a2);
    const uint32_t u2 = lop3<XOR3>(a3, p1, p2);
    const uint32_t u3 = lop3<XOR3>(p3, p5, p7);
    const uint32_t u4 = lop3<XOR3>(p8, p9, p11);
    return lop3<XOR3>(lop3<XOR3>(u1, u2, u3), u4, 0u);
}

// One clock.  INIT = the initialisation mode: z is added to both feedbacks.
template <bool INIT>
__device__ __forceinline__ void clock(uint32_t (&s)[80], uint32_t (&b)[80])
{
    uint32_t fs = f_lfsr(s);
    uint32_t fb = g_nfsr(s[0], b);
    if (INIT) {
        const uint32_t z = output<false>(s, b);
        fs = lop3<XOR2>(fs, z, 0u);
        fb = lop3<XOR2>(fb, z, 0u);
    }
#pragma unroll
    for (int i = 0; i < 79; ++i) {
        s[i] = s[i + 1];
        b[i] = b[i + 1];
    }
    s[79] = fs;
    b[79] = fb;
}

}  // namespace grain

// Cipher traits used by keystream_kernel (keystream.cuh).
struct Grain {
    static constexpr int NSTATE = grain::NSTATE;
    static constexpr bool MSB_FIRST = false;  // spec [15]: keystream packed LSB-first
    // clocks per loop iteration (~45 instructions per clock).  The 80-clock
    // register rotation costs 160/U moves per clock at the back edge; at U = 32
    // ptxas emits them all as IMAD.MOV (FMA pipe), at U = 16 partly as MOV.
    // (U = 8 was dropped after the round-1 sweep: 0.83 of roofline)
    static constexpr int U_DEFAULT = 32, U_ALT0 = 16, U_ALT1 = 16;
    // ROW_MAJOR default: row segments staged in TMEM, two CTAs per SM (+7%
    // over one CTA with smem staging; DESIGN.md sec. 5 Grain)
    static constexpr bool RM_TMEM = true;
    // ...with time segments (~8 per resident warp): a lone Grain warp keeps
    // the ALU only ~70% busy, so a whole-unit tail wave would run slow
    static constexpr bool RM_SEGMENTED = true;
    // ...unless the call has at most one warp-unit per SMSP (the paper's launch
    // shape): lone clock-loop warps then get a writer warp each (rowmajor_ws.cuh;
    // C4 5.82 vs 5.07 Tb/s)
    static constexpr int RM_WS = 1;
    uint32_t s[80], b[80];

    __device__ __forceinline__ void load(const uint32_t* st, uint64_t Gp, uint64_t g)
    {
        const uint32_t* p = opaque(st + g);
#pragma unroll
        for (int i = 0; i < 80; ++i) s[i] = __ldcg(p + uint64_t(i) * Gp);
#pragma unroll
        for (int i = 0; i < 80; ++i) b[i] = __ldcg(p + uint64_t(80 + i) * Gp);
    }
    __device__ __forceinline__ void store(uint32_t* st, uint64_t Gp, uint64_t g) const
    {
        uint32_t* p = opaque(st + g);
#pragma unroll
        for (int i = 0; i < 80; ++i) __stcg(p + uint64_t(i) * Gp, s[i]);
#pragma unroll
        for (int i = 0; i < 80; ++i) __stcg(p + uint64_t(80 + i) * Gp, b[i]);
    }
    __device__ __forceinline__ uint32_t z() const { return grain::output<false>(s, b); }
    // checksum accumulation fused into the output XOR tree
    __device__ __forceinline__ uint32_t z_acc(uint32_t acc) const { return grain::output<true>(s, b, acc); }
    __device__ __forceinline__ void clock() { grain::clock<false>(s, b); }
};

// Initialisation (spec [15]): b_i = key bit i, s_i = IV bit i (i < 64),
// s_64..s_79 = 1, then 160 clocks with z fed back.  Key/IV bits LSB-first.
//   key_s: uint32 [80][Gp], iv_s: uint32 [64][Gp]; state uint32 [161][Gp].
__global__ void __launch_bounds__(128) grain_preclock_kernel(const uint32_t* __restrict__ key_s,
                                                             const uint32_t* __restrict__ iv_s,
                                                             uint32_t* __restrict__ state, uint64_t Gp)
{
    const uint64_t g = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (g >= Gp) return;
    uint32_t s[80], b[80];
#pragma unroll
    for (int i = 0; i < 80; ++i) b[i] = key_s[uint64_t(i) * Gp + g];
#pragma unroll
    for (int i = 0; i < 64; ++i) s[i] = iv_s[uint64_t(i) * Gp + g];
#pragma unroll
    for (int i = 64; i < 80; ++i) s[i] = 0xFFFFFFFFu;
#pragma unroll 1
    for (int c = 0; c < 160; c += 16) {
#pragma unroll
        for (int u = 0; u < 16; ++u) grain::clock<true>(s, b);
    }
#pragma unroll
    for (int i = 0; i < 80; ++i) state[uint64_t(i) * Gp + g] = s[i];
#pragma unroll
    for (int i = 0; i < 80; ++i) state[uint64_t(80 + i) * Gp + g] = b[i];
    state[uint64_t(160) * Gp + g] = 0u;
}

// Fused slicing + initialisation (steps a-1 + a-2 in one kernel): each thread
// slices its 32 instances' key and IV bytes in registers (slice_group32, LSB
// first) straight into the NFSR / LFSR state words -- no sliced copy in HBM,
// no shared memory -- then runs the 160 init clocks.  Group g's keys / IVs
// at raw_k + 320 g / raw_iv + 256 g for g < g_split (16 B aligned), else in
// the zero-padded tail buffers (see m2_init_kernel).
// key / IV rows of the shared-memory staging area (bytes per lane)
constexpr int GI_KSTRIDE = 336, GI_VSTRIDE = 272;
#ifndef GI_UNROLL
#define GI_UNROLL 40
#endif
#ifndef GI_BLOCK
#define GI_BLOCK 128
#endif
constexpr size_t GI_SMEM_BYTES = size_t(GI_BLOCK) * (GI_KSTRIDE + GI_VSTRIDE);  // 19 KB per warp

__global__ void __launch_bounds__(GI_BLOCK) grain_init_kernel(const uint8_t* __restrict__ raw_k,
                                                         const uint8_t* __restrict__ raw_iv,
                                                         const uint8_t* __restrict__ tail_k,
                                                         const uint8_t* __restrict__ tail_iv, uint64_t g_split,
                                                         uint32_t* __restrict__ state, uint64_t Gp)
{
    extern __shared__ __align__(16) uint8_t gi_smem[];
    const uint64_t g = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (g >= Gp) return;  // whole warps (Gp is a multiple of 32)
    const uint32_t lane = threadIdx.x & 31u;
    uint8_t* wk = gi_smem + (threadIdx.x >> 5) * 32 * (GI_KSTRIDE + GI_VSTRIDE);
    uint8_t* wv = wk + 32 * GI_KSTRIDE;
    const uint64_t g0 = g - lane;
    if (g0 + 32 <= g_split) {  // warp-uniform: the warp's 32 groups are contiguous
        stage_warp_groups<320, GI_KSTRIDE>(raw_k + g0 * 320u, wk, lane);
        stage_warp_groups<256, GI_VSTRIDE>(raw_iv + g0 * 256u, wv, lane);
    } else {
        stage_own_group<320, GI_KSTRIDE>(group_src(raw_k, tail_k, g_split, g, 320u), wk, lane);
        stage_own_group<256, GI_VSTRIDE>(group_src(raw_iv, tail_iv, g_split, g, 256u), wv, lane);
    }
    __syncwarp();
    uint32_t s[80], b[80];
    slice_group32<10, 80, false, false>(wk + lane * GI_KSTRIDE, [&](int bit, uint32_t w) { b[bit] = w; });
    slice_group32<8, 64, false, false>(wv + lane * GI_VSTRIDE, [&](int bit, uint32_t w) { s[bit] = w; });
#pragma unroll
    for (int i = 64; i < 80; ++i) s[i] = 0xFFFFFFFFu;
#pragma unroll 1
    // 40 clocks per iteration: the 80-word rotation closes with 160 moves per
    // 40 clocks (4 per clock on the FMA pipe; 10 at 16 clocks per iteration)
    for (int c = 0; c < 160; c += GI_UNROLL) {
#pragma unroll
        for (int u = 0; u < GI_UNROLL; ++u) grain::clock<true>(s, b);
    }
    uint32_t* p = opaque(state + g);
#pragma unroll
    for (int i = 0; i < 80; ++i) __stcg(p + uint64_t(i) * Gp, s[i]);
#pragma unroll
    for (int i = 0; i < 80; ++i) __stcg(p + uint64_t(80 + i) * Gp, b[i]);
    p[uint64_t(160) * Gp] = 0u;
}

}  // namespace bsk
