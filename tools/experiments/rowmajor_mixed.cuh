// rowmajor_mixed.cuh -- EXPERIMENT, NOT BUILT (a measured negative result;
// DESIGN.md sec. 10).  Bit-exact in every Grain GPU test while wired in
// (launch_ks.cuh, option rm_mixed), but Grain C2 ROW_MAJOR ran at 10.74 Tb/s
// against the shipped TMEM + TMA path's 11.47: the store pattern improved as
// the microbenchmark predicted, but the two staging code paths in one CTA
// cost instruction-cache misses (7% no_instruction) and the shared-memory
// half's loads/stores more than the DRAM side gained.
//
// ROW_MAJOR keystream kernel with two staging kinds in one CTA.
//
// A cipher that needs two clock-loop warps per SMSP to keep the ALU busy
// (Grain v1: 0.92 of its roofline in consume vs 0.86 with one) cannot give
// every warp the 64 B of row staging per flush that the DRAM wants: TMEM holds
// 512 columns per lane quarter = 64 B x 1024 rows for ONE warp, and 227 KB of
// shared memory holds 32 B x 1024 rows for at most six.  So the eight
// clock-loop warps of this CTA split: warps 0-3 stage 64 B per row in TMEM
// (all 512 columns of their lane quarter; wide_col permutation, 16x256b
// read-back, one STG.128 per 8 rows x 64 B), warps 4-7 stage 32 B per row in
// shared memory (36 KB each, rows padded to 36 words so both the per-thread
// writes of a transposed block and the lane-quad read-back are bank-conflict
// free) and flush with one STG.64 per 8 rows x 32 B.  All flushes carry an L2
// evict_last hint.  profiles/r2_flush_pattern.log: this mix of pieces writes
// 2.09 TB/s, against 1.53 TB/s when all eight warps flush 32 B per row.
// The clock loop, the 32x32 transposes and the persistent (time segment,
// warp-unit) queue are keystream.cuh's; U = 32 with the z block in registers.
#pragma once
#include <cstdint>

#include "keystream.cuh"

namespace bsk {
namespace mixed {

constexpr int NW = 8;            // clock-loop warps per CTA (two per SMSP)
constexpr int BLOCK = NW * 32;
constexpr int PAD = 36;          // words per (row q, slot k) line of the smem staging
constexpr int SM_WORDS = 32 * 8 * PAD;                 // per smem-staged warp: 36 KB
constexpr size_t SMEM_BYTES = size_t(4) * SM_WORDS * 4;  // 144 KB

// Transpose 32 z words (registers) and write the row words of slot k into the
// padded staging: word (q, k) of lane l at os[(q * 8 + k) * PAD + l].
template <bool MSB_FIRST>
__device__ __forceinline__ void transpose_to_pad(const uint32_t (&z)[32], uint32_t* os, uint32_t k)
{
    constexpr int X = MSB_FIRST ? 7 : 0;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t x[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) x[q] = __byte_perm(z[q ^ X], z[(q + 16) ^ X], h == 0 ? 0x5410 : 0x7632);
        bt_transpose16(x);
#pragma unroll
        for (int q = 0; q < 16; ++q) os[((16 * h + q) * 8 + k) * PAD] = x[q];
    }
}

// Whole 32 B flush of every real row from the padded staging (8 B aligned
// rows): thread t writes 8 bytes (slots 2j, 2j+1, j = t % 4) of the rows of
// groups 16h + t/4 and 16h + t/4 + 8 -- each STG.64 instruction 8 rows x 32 B.
// Bank of word (q*8 + 2j)*36 + la is (8j + la) mod 32: conflict-free.
__device__ __forceinline__ void store_pad_quads(const uint32_t* osw, uint8_t* const* row0s, const uint32_t* nvalids,
                                                uint64_t row_bytes, uint64_t col)
{
    const uint32_t t = laneid_volatile();
    const uint32_t j = t & 3u;
    const uint64_t pol = l2_evict_last_policy();
#pragma unroll 1
    for (uint32_t h = 0; h < 2; ++h) {
        const uint32_t la = 16 * h + (t >> 2), lb = la + 8;
        uint8_t* pa = row0s[la] + col + 8 * j;
        uint8_t* pb = row0s[lb] + col + 8 * j;
        const uint32_t na = nvalids[la], nb = nvalids[lb];
        const uint32_t* sa = osw + (2 * j) * PAD + la;
        const uint32_t* sb = osw + (2 * j) * PAD + lb;
#pragma unroll 4
        for (uint32_t q = 0; q < 32; ++q) {
            const uint32_t a0 = sa[q * 8 * PAD], a1 = sa[q * 8 * PAD + PAD];
            const uint32_t b0 = sb[q * 8 * PAD], b1 = sb[q * 8 * PAD + PAD];
            if (q < na) st64_hint(pa, a0, a1, pol);
            if (q < nb) st64_hint(pb, b0, b1, pol);
            pa = add_fma(pa, row_bytes);
            pb = add_fma(pb, row_bytes);
        }
    }
}

// Partial flush (slots [k_lo, k_hi], item boundaries / 4 B aligned rows):
// this thread's own rows, word by word.
__device__ __forceinline__ void store_pad_partial(const uint32_t* os, uint8_t* row0, uint64_t row_bytes,
                                                  uint32_t nvalid, uint32_t k_lo, uint32_t k_hi, uint64_t col)
{
    uint8_t* p = row0 + col;
    for (uint32_t q = 0; q < nvalid; ++q)
        for (uint32_t k = k_lo; k <= k_hi; ++k)
            __stcs(reinterpret_cast<uint32_t*>(p + q * row_bytes) + (k - k_lo), os[(q * 8 + k) * PAD]);
}

}  // namespace mixed

template <class C>
__global__ void __launch_bounds__(mixed::BLOCK, 1) keystream_rm_mixed_kernel(const __grid_constant__ KsArgs a)
{
    constexpr int U = 32;
    constexpr int KB = ks_block<C, U>();
    static_assert(KB == 1 || 32 % KB == 0, "whole schedule blocks per 32 clocks");
    extern __shared__ __align__(16) uint32_t mx_smem[];  // warps 4..7: [warp - 4][q 32][k 8][PAD]
    __shared__ uint8_t* s_row0[mixed::BLOCK];
    __shared__ uint32_t s_nvalid[mixed::BLOCK];
    __shared__ uint64_t s_b0[mixed::NW];
    __shared__ uint32_t s_nblk[mixed::NW];
    __shared__ uint32_t s_item[mixed::NW];
    __shared__ uint32_t s_tmem;
    (void)tmem_alloc_cta(&s_tmem, true);  // 512 columns: warps 0-3 own their lane quarters

    volatile uint32_t* slot = s_item + (threadIdx.x >> 5);
    next_item(a, slot);
    const uint64_t total = a.units * a.nseg;
    for (;;) {
        uint64_t item = *slot;
        if (item >= total) break;
        uint32_t lane = laneid_volatile();
        uint64_t seg = item / a.units;
        uint64_t w = item - seg * a.units;
        uint64_t g = w * 32u + lane;
        if (seg > 0) {
            if (lane == 0)
                while (ld_acquire(a.flags + w) < seg) __nanosleep(256);
            __syncwarp();
            (void)ld_acquire(a.flags + w);
        }
        const uint64_t clk_begin = seg * a.seg_clocks;
        const uint64_t left = a.nclocks - clk_begin;
        const uint32_t nclk = uint32_t(left < a.seg_clocks ? left : a.seg_clocks);
        C c;
        c.load(a.state, a.Gp, g);
        {
            const uint64_t first = g * 32u;
            const uint32_t nvalid = first >= a.n ? 0u : uint32_t(a.n - first < 32 ? a.n - first : 32);
            s_row0[threadIdx.x] = static_cast<uint8_t*>(a.out) + (nvalid ? first : 0) * a.row_bytes;
            s_nvalid[threadIdx.x] = nvalid;
            if (lane == 0) {
                s_b0[threadIdx.x >> 5] = clk_begin >> 5;
                s_nblk[threadIdx.x >> 5] = nclk >> 5;
            }
            __syncwarp();
        }
#pragma unroll 1
        for (uint32_t blk = 0;; ++blk) {
            const uint32_t wq = tid_volatile() >> 5;
            const uint32_t nblk = *reinterpret_cast<volatile uint32_t*>(&s_nblk[wq]);
            if (blk >= nblk) break;
            uint32_t zr[32];
            static_for<32>([&](auto u) {
                constexpr int J = decltype(u)::value % KB;
                zr[decltype(u)::value] = ks_z<J, KB>(c);
                ks_clock<J, KB>(c);
            });
            const uint32_t wv = tid_volatile() >> 5;  // re-derived: no register held across the clocks
            const uint64_t B = *reinterpret_cast<volatile uint64_t*>(&s_b0[wv]) + blk;
            const uint32_t t = tid_volatile();
            if (wv < 4) {
                // ---- 64 B TMEM staging (lane quarter wv, all 512 columns)
                const uint32_t tm = *reinterpret_cast<volatile uint32_t*>(&s_tmem) + (wv << 21);
                const uint32_t k = uint32_t(B & 15);
                rowmajor_transpose_tmem<C::MSB_FIRST, 16>(zr, tm, wide_col(k));
                if (k == 15 || blk + 1 == nblk) {
                    const uint32_t k_lo = k - (blk < k ? blk : k);
                    const uint64_t col = (B - (k - k_lo)) * 4;
                    if (k_lo == 0 && k == 15 && ((a.row_bytes | col) & 7) == 0 && a.row_bytes < (1ull << 32))
                        rowmajor_store_tmem_wide(tm, s_row0 + (t & ~31u), s_nvalid + (t & ~31u), a.row_bytes, col);
                    else
                        rowmajor_store_tmem_wide_partial(tm, s_row0[t], a.row_bytes, s_nvalid[t], k_lo, k, col);
                }
            } else {
                // ---- 32 B shared-memory staging
                uint32_t* osw = mx_smem + (wv - 4) * mixed::SM_WORDS;
                const uint32_t k = uint32_t(B & 7);
                mixed::transpose_to_pad<C::MSB_FIRST>(zr, osw + laneid_volatile(), k);
                if (k == 7 || blk + 1 == nblk) {
                    __syncwarp();
                    const uint32_t k_lo = k - (blk < k ? blk : k);
                    const uint64_t col = (B - (k - k_lo)) * 4;
                    if (k_lo == 0 && k == 7 && ((a.row_bytes | col) & 7) == 0 && a.row_bytes < (1ull << 32))
                        mixed::store_pad_quads(osw, s_row0 + (t & ~31u), s_nvalid + (t & ~31u), a.row_bytes, col);
                    else
                        mixed::store_pad_partial(osw + laneid_volatile(), s_row0[t], a.row_bytes, s_nvalid[t], k_lo,
                                                 k, col);
                    __syncwarp();
                }
            }
        }
        // re-derive the item context (kept out of registers during the loop)
        item = *slot;
        lane = laneid_volatile();
        seg = item / a.units;
        w = item - seg * a.units;
        g = w * 32u + lane;
        c.store(a.state, a.Gp, g);
        if (seg + 1 != a.nseg) {
            __threadfence();
            __syncwarp();
            if (lane == 0) st_release(a.flags + w, uint32_t(seg + 1));
        }
        next_item(a, slot);
    }
    tmem_dealloc_cta(*reinterpret_cast<volatile uint32_t*>(&s_tmem), true);
}

}  // namespace bsk
