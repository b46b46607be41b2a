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
//   SubBytes: 16 x the Boyar-Peralta depth-16 S-box circuit (113 gates:
//            32 AND, 81 XOR/XNOR; verified against the S-box table)
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

// Boyar-Peralta S-box circuit on one byte: u[0] = MSB ... u[7] = LSB (in place).
__device__ __forceinline__ void sbox(uint32_t& U0, uint32_t& U1, uint32_t& U2, uint32_t& U3, uint32_t& U4,
                                     uint32_t& U5, uint32_t& U6, uint32_t& U7)
{
    const uint32_t T1 = U0 ^ U3, T2 = U0 ^ U5, T3 = U0 ^ U6, T4 = U3 ^ U5, T5 = U4 ^ U6;
    const uint32_t T6 = T1 ^ T5, T7 = U1 ^ U2, T8 = U7 ^ T6, T9 = U7 ^ T7, T10 = T6 ^ T7;
    const uint32_t T11 = U1 ^ U5, T12 = U2 ^ U5, T13 = T3 ^ T4, T14 = T6 ^ T11, T15 = T5 ^ T11;
    const uint32_t T16 = T5 ^ T12, T17 = T9 ^ T16, T18 = U3 ^ U7, T19 = T7 ^ T18, T20 = T1 ^ T19;
    const uint32_t T21 = U6 ^ U7, T22 = T7 ^ T21, T23 = T2 ^ T22, T24 = T2 ^ T10, T25 = T20 ^ T17;
    const uint32_t T26 = T3 ^ T16, T27 = T1 ^ T12;
    const uint32_t D = U7;
    const uint32_t M1 = T13 & T6, M2 = T23 & T8, M3 = T14 ^ M1, M4 = T19 & D, M5 = M4 ^ M1;
    const uint32_t M6 = T3 & T16, M7 = T22 & T9, M8 = T26 ^ M6, M9 = T20 & T17, M10 = M9 ^ M6;
    const uint32_t M11 = T1 & T15, M12 = T4 & T27, M13 = M12 ^ M11, M14 = T2 & T10, M15 = M14 ^ M11;
    const uint32_t M16 = M3 ^ M2, M17 = M5 ^ T24, M18 = M8 ^ M7, M19 = M10 ^ M15, M20 = M16 ^ M13;
    const uint32_t M21 = M17 ^ M15, M22 = M18 ^ M13, M23 = M19 ^ T25, M24 = M22 ^ M23, M25 = M22 & M20;
    const uint32_t M26 = M21 ^ M25, M27 = M20 ^ M21, M28 = M23 ^ M25, M29 = M28 & M27, M30 = M26 & M24;
    const uint32_t M31 = M20 & M23, M32 = M27 & M31, M33 = M27 ^ M25, M34 = M21 & M22, M35 = M24 & M34;
    const uint32_t M36 = M24 ^ M25, M37 = M21 ^ M29, M38 = M32 ^ M33, M39 = M23 ^ M30, M40 = M35 ^ M36;
    const uint32_t M41 = M38 ^ M40, M42 = M37 ^ M39, M43 = M37 ^ M38, M44 = M39 ^ M40, M45 = M42 ^ M41;
    const uint32_t M46 = M44 & T6, M47 = M40 & T8, M48 = M39 & D, M49 = M43 & T16, M50 = M38 & T9;
    const uint32_t M51 = M37 & T17, M52 = M42 & T15, M53 = M45 & T27, M54 = M41 & T10, M55 = M44 & T13;
    const uint32_t M56 = M40 & T23, M57 = M39 & T19, M58 = M43 & T3, M59 = M38 & T22, M60 = M37 & T20;
    const uint32_t M61 = M42 & T1, M62 = M45 & T4, M63 = M41 & T2;
    const uint32_t L0 = M61 ^ M62, L1 = M50 ^ M56, L2 = M46 ^ M48, L3 = M47 ^ M55, L4 = M54 ^ M58;
    const uint32_t L5 = M49 ^ M61, L6 = M62 ^ L5, L7 = M46 ^ L3, L8 = M51 ^ M59, L9 = M52 ^ M53;
    const uint32_t L10 = M53 ^ L4, L11 = M60 ^ L2, L12 = M48 ^ M51, L13 = M50 ^ L0, L14 = M52 ^ M61;
    const uint32_t L15 = M55 ^ L1, L16 = M56 ^ L0, L17 = M57 ^ L1, L18 = M58 ^ L8, L19 = M63 ^ L4;
    const uint32_t L20 = L0 ^ L1, L21 = L1 ^ L7, L22 = L3 ^ L12, L23 = L18 ^ L2, L24 = L15 ^ L9;
    const uint32_t L25 = L6 ^ L10, L26 = L7 ^ L9, L27 = L8 ^ L10, L28 = L11 ^ L14, L29 = L11 ^ L17;
    U0 = L6 ^ L24;
    U1 = ~(L16 ^ L26);
    U2 = ~(L19 ^ L28);
    U3 = L6 ^ L21;
    U4 = L20 ^ L22;
    U5 = L25 ^ L29;
    U6 = ~(L13 ^ L27);
    U7 = ~(L6 ^ L23);
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

// xtime on one byte held MSB-first in v[0..7]: result bit i (significance)
// is v<<1 with 0x1b folded in where the old MSB was set.
__device__ __forceinline__ void xtime(const uint32_t (&v)[8], uint32_t (&o)[8])
{
    // significance k <-> index 7-k
    o[7] = v[0];          // bit0 = old bit7
    o[6] = v[7] ^ v[0];   // bit1 = old bit0 ^ bit7
    o[5] = v[6];          // bit2 = old bit1
    o[4] = v[5] ^ v[0];   // bit3 = old bit2 ^ bit7
    o[3] = v[4] ^ v[0];   // bit4 = old bit3 ^ bit7
    o[2] = v[3];          // bit5 = old bit4
    o[1] = v[2];          // bit6 = old bit5
    o[0] = v[1];          // bit7 = old bit6
}

// MixColumns (FIPS-197 5.1.3) + AddRoundKey with round-key row `k` (masks).
__device__ __forceinline__ void mix_columns_ark(uint32_t (&s)[128], const uint32_t* k)
{
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        uint32_t a[4][8];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int b = 0; b < 8; ++b) a[i][b] = s[8 * (4 * c + i) + b];
        uint32_t t[8];
#pragma unroll
        for (int b = 0; b < 8; ++b) t[b] = a[0][b] ^ a[1][b] ^ a[2][b] ^ a[3][b];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            uint32_t u[8], x[8];
#pragma unroll
            for (int b = 0; b < 8; ++b) u[b] = a[i][b] ^ a[(i + 1) & 3][b];
            xtime(u, x);
#pragma unroll
            for (int b = 0; b < 8; ++b) s[8 * (4 * c + i) + b] = a[i][b] ^ t[b] ^ x[b] ^ k[8 * (4 * c + i) + b];
        }
    }
}

__device__ __forceinline__ void add_round_key(uint32_t (&s)[128], const uint32_t* k)
{
#pragma unroll
    for (int i = 0; i < 128; ++i) s[i] ^= k[i];
}

// Counter block for encryption index T (warp-uniform) plus round-0 key:
// s = (base + T mod 2^128) ^ K0.  base is this thread's sliced initial
// counter (128 words in shared memory, [b][thread] with stride `st`).
// Bit b has significance 127 - b; the carry ripples from word 127 up.
__device__ __forceinline__ void counter_block(uint32_t (&s)[128], const uint32_t* base, int st, uint64_t T,
                                              const RoundKeys& rk)
{
    uint32_t c = 0u;
#pragma unroll
    for (int p = 0; p < 128; ++p) {
        const int b = 127 - p;
        const uint32_t x = base[b * st];
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

__global__ void aes_key_expand_kernel(const uint8_t* __restrict__ key, uint32_t* __restrict__ masks)
{
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    uint8_t w[176];
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
    for (int r = 0; r < 11; ++r)
        for (int b = 0; b < 128; ++b)
            masks[r * 128 + b] = ((w[16 * r + b / 8] >> (7 - b % 8)) & 1u) ? 0xFFFFFFFFu : 0u;
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
__global__ void __launch_bounds__(128, 1) aes_ctr_kernel(const KsArgs a, const __grid_constant__ aes::RoundKeys rk)
{
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
            aes::counter_block(s, base, 128, T0 + e, rk);
            aes::encrypt(s, rk);
            if (LAYOUT == L_CHECKSUM) {
#pragma unroll
                for (int b = 0; b < 128; ++b) acc ^= s[b];
            } else if (LAYOUT == L_SLICED) {
                if (g < a.G) {
                    uint32_t* o = static_cast<uint32_t*>(a.out) + (bit_begin + uint64_t(e) * 128) * a.G + g;
#pragma unroll
                    for (int b = 0; b < 128; ++b) __stcs(o + uint64_t(b) * a.G, s[b] & m);
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

}  // namespace bsk
