// aes.cuh -- bitsliced AES-128 in counter mode for sm_100a (SURVEY sec. 8(f)
// NEXT-2).
//
// PAPER.md:288-338 (sec. 2.3.2, Fig. 3): AES-CTR as a PRNG -- counter blocks,
// one 128-bit output block per counter value, fully parallel; PAPER.md:
// 456-460 and 757-760: the paper's bitsliced AES kernel, "limited" by its
// bitsliced S-box; "different counter values ... with a
// unique key".  Cipher: FIPS-197 (ref [35]).
//
// Layout: one thread = 32 counter streams (instances); the 128-bit block is
// 128 slice words, word b = bit b of the block for 32 lanes, bit b = bit
// (7 - b%8) of byte b/8 (FIPS-197 bit order), so byte j = words 8j..8j+7 with
// word 8j its most significant bit.  All instances share one key, so every
// round-key bit is a warp-uniform constant: the 11 x 128 round-key masks
// (0 / ~0) are passed as a kernel parameter and ptxas folds AddRoundKey into
// LOP3s with a constant-bank operand.
//
// Per encryption (32 blocks = 4096 keystream bits per thread):
//   counter: x = base + T (128-bit big-endian add of the warp-uniform block
//            index T to the sliced initial counters, ripple carry), fused with
//            round-0 AddRoundKey                                  ~256 LOP3
//   SubBytes: 16 x the Boyar-Peralta depth-16 S-box circuit as 84 LOP3s
//            (tools/lut3_map.py; 113 two-input gates originally)
//   ShiftRows: register renaming; MixColumns + AddRoundKey: XOR trees.
// AES-CTR has no state carried between blocks: work items of one instance in
// different time segments are independent (no segment flags).
#pragma once
#include <cstdint>

#include "keystream.cuh"

namespace bsk {
namespace aes {

constexpr int NSTATE = 128;  // sliced initial counter block per group

// Round-key masks: m[r][b] = ~0 if bit b of round key r is 1, else 0.
struct RoundKeys {
    uint32_t m[11][128];
};

// Round keys live in constant memory, one slot per AES handle: the key
// expansion kernel writes the masks to device memory and a stream-ordered
// device-to-device cudaMemcpyToSymbolAsync moves them into the handle's slot,
// so a rekey never waits on the host.  The keystream kernels read them with a
// warp-uniform (slot, round) index -- uniform constant loads (LDCU) feeding
// the AddRoundKey LOP3s.  11 slots x 5.5 KB fit the 64 KB constant bank.
constexpr int RK_SLOTS = 11;
__constant__ RoundKeys c_rk[RK_SLOTS];

// AES S-box on one byte held MSB-first in 8 slice words (in place): the
// Boyar-Peralta depth-16 circuit (113 two-input gates) mapped onto 84
// three-input LOP3s by tools/lut3_map.py (cut enumeration + area recovery),
// verified there against the FIPS-197 S-box on all 256 inputs.
__device__ __forceinline__ void sbox(uint32_t& U0, uint32_t& U1, uint32_t& U2, uint32_t& U3, uint32_t& U4,
                                     uint32_t& U5, uint32_t& U6, uint32_t& U7)
{
    uint32_t S0, S1, S2, S3, S4, S5, S6, S7;
#include "aes_sbox_lop3.inc"
    U0 = S0;
    U1 = S1;
    U2 = S2;
    U3 = S3;
    U4 = S4;
    U5 = S5;
    U6 = S6;
    U7 = S7;
}

__device__ __forceinline__ void sub_bytes(uint32_t (&s)[128])
{
#pragma unroll
    for (int j = 0; j < 16; ++j)
        sbox(s[8 * j + 0], s[8 * j + 1], s[8 * j + 2], s[8 * j + 3], s[8 * j + 4], s[8 * j + 5], s[8 * j + 6],
             s[8 * j + 7]);
}

// byte j = r + 4c of the result takes byte r + 4((c + r) % 4)  (FIPS-197 5.1.2)
__device__ __forceinline__ void shift_rows(uint32_t (&s)[128])
{
    uint32_t t[128];
#pragma unroll
    for (int j = 0; j < 16; ++j) {
        const int r = j & 3, c = j >> 2;
        const int src = r + 4 * ((c + r) & 3);
#pragma unroll
        for (int k = 0; k < 8; ++k) t[8 * j + k] = s[8 * src + k];
    }
#pragma unroll
    for (int i = 0; i < 128; ++i) s[i] = t[i];
}

// MixColumns (FIPS-197 5.1.3) + AddRoundKey with round-key row `k` (masks):
// per column, out_i = 2a_i ^ 3a_{i+1} ^ a_{i+2} ^ a_{i+3} ^ k, a GF(2)-linear
// map of the column's 32 bit words plus one key word per output.  The
// program is tools/mc_xor3.py's three-input-XOR circuit (greedy common-
// subexpression search over 2- and 3-input XOR gates, verified there by
// simulation and here by the FIPS/SP 800-38A vectors): 84 LOP3 per column,
// against 96 for the u_i = a_i ^ a_{i+1} form (32 XOR2 for u, then
// a_{i+1} ^ u_{i+2} ^ xtime(u_i) ^ k as two LOP3 per output bit).
__device__ __forceinline__ uint32_t x2(uint32_t a, uint32_t b) { return lop3<0x3Cu>(a, b, 0u); }
__device__ __forceinline__ uint32_t x3(uint32_t a, uint32_t b, uint32_t c) { return lop3<0x96u>(a, b, c); }
__device__ __forceinline__ void mix_columns_ark(uint32_t (&s)[128], const uint32_t* k)
{
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        uint32_t a[32], o[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) a[j] = s[32 * c + j];
        const uint32_t* kk = k + 32 * c;
#include "aes_mc_lop3.inc"
#pragma unroll
        for (int j = 0; j < 32; ++j) s[32 * c + j] = o[j];
    }
}

__device__ __forceinline__ void add_round_key(uint32_t (&s)[128], const uint32_t* k)
{
#pragma unroll
    for (int i = 0; i < 128; ++i) s[i] ^= k[i];
}

// Counter block for encryption index T (warp-uniform) plus round-0 key:
// s = (base + T mod 2^128) ^ K0.  base is this thread's sliced initial
// counter (128 words in shared memory, [b][thread] with stride `st`, as a
// shared-window address).  The loads are volatile: hoisted out of the
// encryption loop, the 128 loop-invariant words spilled 272 B of stack.
// Bit b has significance 127 - b; the carry ripples from word 127 up.
__device__ __forceinline__ uint32_t lds_volatile(uint32_t saddr)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(saddr));
    return v;
}
__device__ __forceinline__ void counter_block(uint32_t (&s)[128], uint32_t base, int st, uint64_t T,
                                              const RoundKeys& rk)
{
    uint32_t c = 0u;
#pragma unroll
    for (int p = 0; p < 128; ++p) {
        const int b = 127 - p;
        const uint32_t x = lds_volatile(base + 4u * uint32_t(b * st));
        const uint32_t tb = p < 64 ? (uint32_t)0 - (uint32_t)((T >> p) & 1u) : 0u;  // warp-uniform
        s[b] = x ^ c ^ (tb ^ rk.m[0][b]);
        c = (x & c) | ((x | c) & tb);  // majority(x, tb, c)
    }
}

// Rounds 1..10.  The round is a loop (not unrolled): one fully unrolled
// round is ~1750 instructions (28 KB of SASS) and fits the instruction cache,
// ten of them (300 KB) do not -- ncu showed `no_instruction` as the dominant
// stall with the rounds unrolled.  Round keys are read with a warp-uniform
// runtime index from the kernel-parameter constant bank.
// Block-lane layout (ROW_MAJOR kernel below): the 32 lanes of a thread are 32
// CONSECUTIVE blocks V + j of ONE instance.  V is the 128-bit big-endian block
// value of lane 0 (V[0] most significant).  With c = V mod 32, H = V >> 5:
//   significance 0..4 of block j = bits of (c + j) mod 32 -> the lane patterns
//     0xAAAAAAAA, 0xCCCCCCCC, ... rotated right by c;
//   significance 5..127 = bits of H, or of H + 1 in the lanes j >= 32 - c that
//     carried out of the low five bits.
// Round key 0 is folded in: the K0 bits >= 5 are XORed into H and H + 1 before
// the per-bit masks are extracted.
template <int Q>
__device__ __forceinline__ uint32_t bit_mask(uint32_t w)
{
    // 0 or ~0 = bit Q of w: the shift on the FMA pipe (IMAD.SHL), the sign
    // broadcast on the ALU pipe
    return uint32_t(int32_t(shl_fma<31 - Q>(w)) >> 31);
}

__device__ __forceinline__ void counter_block_lanes(uint32_t (&s)[128], const uint32_t (&V)[4], const RoundKeys& rk,
                                                    const uint32_t (&K0hi)[4])
{
    const uint32_t c = V[3] & 31u;
    const uint32_t carry = c ? (0xFFFFFFFFu << (32 - c)) : 0u;
    uint32_t H[4], H1[4];
    H[3] = (V[3] >> 5) | (V[2] << 27);
    H[2] = (V[2] >> 5) | (V[1] << 27);
    H[1] = (V[1] >> 5) | (V[0] << 27);
    H[0] = V[0] >> 5;
    // bits >= 27 of H and H + 1 agree unless bits 0..26 of H are all ones
    const bool hi_equal = (H[3] & 0x07FFFFFFu) != 0x07FFFFFFu;
    uint32_t cy = 1u;
#pragma unroll
    for (int w = 3; w >= 0; --w) {
        H1[w] = H[w] + cy;
        cy = (cy && H1[w] == 0u) ? 1u : 0u;
    }
#pragma unroll
    for (int w = 0; w < 4; ++w) {
        H[w] ^= K0hi[w];
        H1[w] ^= K0hi[w];
    }
    constexpr uint32_t P0[5] = {0xAAAAAAAAu, 0xCCCCCCCCu, 0xF0F0F0F0u, 0xFF00FF00u, 0xFFFF0000u};
#pragma unroll
    for (int p = 0; p < 5; ++p) s[127 - p] = __funnelshift_r(P0[p], P0[p], c) ^ rk.m[0][127 - p];
    // lanes j >= 32 - c carried out of the low five bits: they see H + 1
    static_for<27>([&](auto qq) {
        constexpr int q = decltype(qq)::value;
        s[127 - 5 - q] = sel_imm_var(carry, bit_mask<q>(H1[3]), bit_mask<q>(H[3]));
    });
    if (hi_equal) {  // the common case: one mask per bit, no select
        static_for<96>([&](auto qq) {
            constexpr int q = decltype(qq)::value + 27;
            s[127 - 5 - q] = bit_mask<q & 31>(H[3 - (q >> 5)]);
        });
    } else {
        static_for<96>([&](auto qq) {
            constexpr int q = decltype(qq)::value + 27;
            s[127 - 5 - q] = sel_imm_var(carry, bit_mask<q & 31>(H1[3 - (q >> 5)]), bit_mask<q & 31>(H[3 - (q >> 5)]));
        });
    }
}

__device__ __forceinline__ void encrypt(uint32_t (&s)[128], const RoundKeys& rk)
{
#pragma unroll 1
    for (int r = 1; r < 10; ++r) {
        sub_bytes(s);
        shift_rows(s);
        mix_columns_ark(s, rk.m[r]);
    }
    sub_bytes(s);
    shift_rows(s);
    add_round_key(s, rk.m[10]);
}

// Key expansion (FIPS-197 5.2) on the device: one thread, writes the 11 x 128
// round-key masks.  S-box values come from the same bitsliced circuit (on
// all-0 / all-1 words), so no table is needed.
__device__ __forceinline__ uint8_t sbox_byte(uint8_t x)
{
    uint32_t u[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) u[k] = ((x >> (7 - k)) & 1u) ? 0xFFFFFFFFu : 0u;
    sbox(u[0], u[1], u[2], u[3], u[4], u[5], u[6], u[7]);
    uint8_t r = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) r |= uint8_t((u[k] & 1u) << (7 - k));
    return r;
}

// One warp: lane 0 runs the (sequential) schedule into shared memory, then the
// 32 lanes expand the 1408 mask words with coalesced stores (the single-thread
// version spent ~37 us on local-memory traffic and serial stores).
__global__ void __launch_bounds__(32) aes_key_expand_kernel(const uint8_t* __restrict__ key,
                                                            uint32_t* __restrict__ masks)
{
    __shared__ uint8_t w[176];
    if (blockIdx.x != 0) return;
    if (threadIdx.x == 0) {
    for (int i = 0; i < 16; ++i) w[i] = key[i];
    uint8_t rcon = 1;
    for (int i = 4; i < 44; ++i) {
        uint8_t t0 = w[4 * i - 4], t1 = w[4 * i - 3], t2 = w[4 * i - 2], t3 = w[4 * i - 1];
        if (i % 4 == 0) {
            const uint8_t r0 = sbox_byte(t1) ^ rcon, r1 = sbox_byte(t2), r2 = sbox_byte(t3), r3 = sbox_byte(t0);
            t0 = r0;
            t1 = r1;
            t2 = r2;
            t3 = r3;
            rcon = uint8_t((rcon << 1) ^ ((rcon & 0x80) ? 0x1b : 0));
        }
        w[4 * i + 0] = w[4 * i - 16] ^ t0;
        w[4 * i + 1] = w[4 * i - 15] ^ t1;
        w[4 * i + 2] = w[4 * i - 14] ^ t2;
        w[4 * i + 3] = w[4 * i - 13] ^ t3;
    }
    }
    __syncwarp();
    for (int i = threadIdx.x; i < 11 * 128; i += 32)
        masks[i] = ((w[i / 8] >> (7 - i % 8)) & 1u) ? 0xFFFFFFFFu : 0u;  // round i/128, bit i%128
}

}  // namespace aes

// ---------------------------------------------------------------------------
// The AES-CTR keystream kernel: persistent, items = (time segment, warp-unit),
// no dependencies between items.  `a.nclocks` / `a.seg_clocks` / `a.t0` are
// in keystream BITS (multiples of 128; segments multiples of 256).
//   CHECKSUM : per-item XOR of the output words, combined by atomicXor into
//              state row 128; the last item of a unit (per-unit counter in
//              a.flags) applies fmix64 and adds the warp sum to *out.
//   SLICED   : out[t][g], 128 coalesced stores per encryption.
//   ROW_MAJOR: the 128 output words are four 32x32 bit tiles already in
//              registers: transposed in place, staged per 32 B sector in smem
//              (two encryptions fill a sector) and written as 16 B stores.
// ---------------------------------------------------------------------------
template <int LAYOUT>
__global__ void __launch_bounds__(128, 2) aes_ctr_kernel(const __grid_constant__ KsArgs a, int rk_slot)
{
    const aes::RoundKeys& rk = aes::c_rk[rk_slot];
    constexpr int NW = 4;
    extern __shared__ uint32_t aes_smem[];  // base counters [128][128 threads] (+ ROW_MAJOR sector buffers)
    __shared__ uint32_t s_item[NW];
    uint32_t* base = aes_smem + threadIdx.x;  // stride 128
    uint32_t* os = aes_smem + 128 * 128 + (threadIdx.x >> 5) * OS_WORDS + (threadIdx.x & 31);
    volatile uint32_t* slot = s_item + (threadIdx.x >> 5);
    next_item(a, slot);
    const uint64_t total = a.units * a.nseg;

    for (;;) {
        const uint64_t item = *slot;
        if (item >= total) break;
        const uint32_t lane = threadIdx.x & 31u;
        const uint64_t seg = item / a.units;
        const uint64_t w = item - seg * a.units;
        const uint64_t g = w * 32u + lane;
        const uint64_t bit_begin = seg * a.seg_clocks;  // call-relative
        const uint64_t left = a.nclocks - bit_begin;
        const uint32_t nenc = uint32_t((left < a.seg_clocks ? left : a.seg_clocks) >> 7);
        {
            const uint32_t* src = opaque(a.state + g);
#pragma unroll 8
            for (int b = 0; b < 128; ++b) base[b * 128] = __ldcg(src + uint64_t(b) * a.Gp);
        }
        __syncwarp();
        const uint64_t T0 = (a.t0 + bit_begin) >> 7;  // block index of the first encryption
        uint32_t acc = 0;
        const uint32_t m = lane_mask(a, g);
        uint64_t first = g * 32u;
        const uint32_t nvalid = first >= a.n ? 0u : uint32_t(a.n - first < 32 ? a.n - first : 32);
        uint8_t* row0 = static_cast<uint8_t*>(a.out) + (nvalid ? first : 0) * a.row_bytes;

#pragma unroll 1
        for (uint32_t e = 0; e < nenc; ++e) {
            uint32_t s[128];
            aes::counter_block(s, static_cast<uint32_t>(__cvta_generic_to_shared(base)), 128, T0 + e, rk);
            aes::encrypt(s, rk);
            if (LAYOUT == L_CHECKSUM) {
#pragma unroll
                for (int b = 0; b < 128; ++b) acc ^= s[b];
            } else if (LAYOUT == L_SLICED) {
                if (g < a.G) {
                    // one running pointer (IMAD.WIDE on the FMA pipe): 128
                    // precomputed addresses spilled
                    uint8_t* o = reinterpret_cast<uint8_t*>(static_cast<uint32_t*>(a.out) +
                                                            (bit_begin + uint64_t(e) * 128) * a.G + g);
                    const uint64_t stride = a.G * 4;
#pragma unroll
                    for (int b = 0; b < 128; ++b) {
                        __stcs(reinterpret_cast<uint32_t*>(o), s[b] & m);
                        o = add_fma(o, stride);
                    }
                }
            } else {
                // four 32-bit tiles: row t of tile k is bit 32k + (t ^ 7) (MSB-first bytes)
                const uint64_t B0 = (bit_begin >> 5) + uint64_t(e) * 4;  // call-relative 32-bit block
#pragma unroll
                for (int k = 0; k < 4; ++k) {
#pragma unroll
                    for (int h = 0; h < 2; ++h) {
                        uint32_t x[16];
#pragma unroll
                        for (int q = 0; q < 16; ++q)
                            x[q] = __byte_perm(s[32 * k + (q ^ 7)], s[32 * k + ((q + 16) ^ 7)], h == 0 ? 0x5410 : 0x7632);
                        bt_transpose16(x);
                        const uint32_t slot8 = uint32_t((B0 + k) & 7);
#pragma unroll
                        for (int q = 0; q < 16; ++q) os[((16 * h + q) * 8 + slot8) * 32] = x[q];
                    }
                }
                const uint32_t k_hi = uint32_t((B0 + 3) & 7);
                if (k_hi == 7 || e + 1 == nenc) {
                    const uint32_t k_lo = (k_hi == 7 && e > 0 && ((B0 & 7) == 4)) ? 0u : uint32_t(B0 & 7);
                    rowmajor_store(os, row0, a.row_bytes, nvalid, k_lo, k_hi, (B0 + 3 - (k_hi - k_lo)) * 4);
                }
            }
        }
        if (LAYOUT == L_CHECKSUM) {
            acc &= m;
            if (a.nseg == 1) {
                uint64_t v = g < a.G ? fmix64(uint64_t(acc) ^ ((a.g_base + g) * 0x9E3779B97F4A7C15ull) ^
                                              (a.t0 * 0xBF58476D1CE4E5B9ull))
                                     : 0ull;
#pragma unroll
                for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, off);
                if (lane == 0) atomicAdd(static_cast<unsigned long long*>(a.out), (unsigned long long)v);
            } else {
                uint32_t* accp = a.state + uint64_t(aes::NSTATE) * a.Gp + g;
                atomicXor(accp, acc);
                __threadfence();
                __syncwarp();
                uint32_t done = 0;
                if (lane == 0) done = atomicAdd(a.flags + w, 1u);
                done = __shfl_sync(0xFFFFFFFFu, done, 0);
                if (done + 1 == a.nseg) {  // last item of this unit: finish its groups
                    __threadfence();
                    const uint32_t full = __ldcg(accp);
                    uint64_t v = g < a.G ? fmix64(uint64_t(full) ^ ((a.g_base + g) * 0x9E3779B97F4A7C15ull) ^
                                                  (a.t0 * 0xBF58476D1CE4E5B9ull))
                                         : 0ull;
#pragma unroll
                    for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, off);
                    if (lane == 0) atomicAdd(static_cast<unsigned long long*>(a.out), (unsigned long long)v);
                }
            }
        }
        next_item(a, slot);
    }
}

// ---------------------------------------------------------------------------
// ROW_MAJOR in the block-lane layout: thread = ONE instance, lane j = block
// V + j.  After the rounds, transposing the four 32x32 tiles in registers
// leaves block j's 16 bytes in s[j], s[32+j], s[64+j], s[96+j]: one 16 B
// store per block, 512 contiguous bytes of the instance's row per
// encryption -- whole sectors with no shared-memory staging.  Used when a call
// has >= 32 blocks per instance (otherwise most lanes would be wasted).
// Work items: (time segment of whole 4096-bit encryptions, 32-instance warp);
// `a.units` counts warps here.  A warp's 32 instances are group w, so each
// thread reads its initial counter back out of the group's sliced state rows
// (bit `lane` of row b = FIPS bit b of its counter block).
// ---------------------------------------------------------------------------
__global__ void __launch_bounds__(128, 2) aes_ctr_rowmajor_lanes_kernel(const __grid_constant__ KsArgs a, int rk_slot)
{
    const aes::RoundKeys& rk = aes::c_rk[rk_slot];
    __shared__ uint32_t s_item[4];
    volatile uint32_t* slot = s_item + (threadIdx.x >> 5);
    next_item(a, slot);
    const uint64_t total = a.units * a.nseg;
    uint32_t K0hi[4];  // bits >= 5 of round key 0 as a 123-bit value (H's alignment)
    {
        uint32_t K[4] = {0, 0, 0, 0};
#pragma unroll
        for (int b = 0; b < 128; ++b) K[b >> 5] |= (rk.m[0][b] & 1u) << (31 - (b & 31));
        K0hi[3] = (K[3] >> 5) | (K[2] << 27);
        K0hi[2] = (K[2] >> 5) | (K[1] << 27);
        K0hi[1] = (K[1] >> 5) | (K[0] << 27);
        K0hi[0] = K[0] >> 5;
    }
    for (;;) {
        const uint64_t item = *slot;
        if (item >= total) break;
        const uint32_t lane = threadIdx.x & 31u;
        const uint64_t seg = item / a.units;
        const uint64_t w = item - seg * a.units;
        const uint64_t inst = w * 32u + lane;
        const bool real = inst < a.n;
        const uint64_t bit_begin = seg * a.seg_clocks;
        const uint64_t left = a.nclocks - bit_begin;
        const uint64_t nblocks = (left < a.seg_clocks ? left : a.seg_clocks) >> 7;
        // V = ctr_inst + first block index of this item (128-bit big-endian),
        // the counter gathered from the sliced state (warp-uniform addresses)
        uint32_t V[4] = {0, 0, 0, 0};
        {
            const uint32_t* src = opaque(a.state + w);
#pragma unroll
            for (int b = 0; b < 128; ++b)
                V[b >> 5] |= ((__ldcg(src + uint64_t(b) * a.Gp) >> lane) & 1u) << (31 - (b & 31));
        }
        {
            const uint64_t T = (a.t0 + bit_begin) >> 7;
            uint64_t lo = (uint64_t(V[2]) << 32) | V[3];
            uint64_t hi = (uint64_t(V[0]) << 32) | V[1];
            const uint64_t nlo = lo + T;
            hi += (nlo < lo) ? 1u : 0u;
            lo = nlo;
            V[0] = uint32_t(hi >> 32);
            V[1] = uint32_t(hi);
            V[2] = uint32_t(lo >> 32);
            V[3] = uint32_t(lo);
        }
        uint8_t* row = static_cast<uint8_t*>(a.out) + (real ? inst : 0) * a.row_bytes + (bit_begin >> 3);
#pragma unroll 1
        for (uint64_t blk = 0; blk < nblocks; blk += 32) {
            uint32_t s[128];
            aes::counter_block_lanes(s, V, rk, K0hi);
            aes::encrypt(s, rk);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                uint32_t x0[16], x1[16];
#pragma unroll
                for (int q = 0; q < 16; ++q) {
                    const uint32_t lo = s[32 * k + (q ^ 7)], hi = s[32 * k + ((q + 16) ^ 7)];
                    x0[q] = __byte_perm(lo, hi, 0x5410);
                    x1[q] = __byte_perm(lo, hi, 0x7632);
                }
                bt_transpose16(x0);
                bt_transpose16(x1);
#pragma unroll
                for (int q = 0; q < 16; ++q) {
                    s[32 * k + q] = x0[q];
                    s[32 * k + 16 + q] = x1[q];
                }
            }
            const uint64_t nb = nblocks - blk < 32 ? nblocks - blk : 32;
            if (real) {
                uint4* dst = reinterpret_cast<uint4*>(row + blk * 16);
                if (nb == 32) {
#pragma unroll
                    for (int j = 0; j < 32; ++j) __stcs(dst + j, make_uint4(s[j], s[32 + j], s[64 + j], s[96 + j]));
                } else {
#pragma unroll
                    for (int j = 0; j < 32; ++j)
                        if (uint64_t(j) < nb) __stcs(dst + j, make_uint4(s[j], s[32 + j], s[64 + j], s[96 + j]));
                }
            }
            // V += 32
            const uint32_t v3 = V[3] + 32u;
            uint32_t cy = v3 < V[3] ? 1u : 0u;
            V[3] = v3;
#pragma unroll
            for (int k = 2; k >= 0; --k) {
                const uint32_t t = V[k] + cy;
                cy = (cy && t == 0u) ? 1u : 0u;
                V[k] = t;
            }
        }
        next_item(a, slot);
    }
}

}  // namespace bsk
