// grain_split.cuh -- EXPERIMENT, NOT BUILT (a measured negative result kept
// for the record).  Bit-exact in every Grain GPU test while
// it was wired in (cipher_grain.cu, option rm_split), but slower than the
// shipped path: C2 ROW_MAJOR 9.79 vs 11.46 Tb/s, paper shape 5.70 vs 5.86 --
// the NFSR warp ran at ~120 cycles per clock beside its LFSR + writer warp
// instead of the ~75 the probe (tools/microbench/grain_split_probe.cu) showed
// for it alone.
//
// Grain v1 ROW_MAJOR with one warp-unit split over two warps of the same SMSP.
//
// Why: the ROW_MAJOR store pattern needs 64 B per row per flush (DESIGN.md
// sec. 5 "ROW_MAJOR output"), i.e. all 512 TMEM columns of a lane quarter for
// ONE warp-unit per SMSP; but a lone warp running all of Grain issues its
// 37-LOP3 clock at only ~0.7 of the ALU (ptxas's schedule leaves dependent
// LOP3s adjacent).  Grain's LFSR (Fig. 4: s, feedback f) does
// not depend on the NFSR, so the unit's two registers go to two warps:
//
//   N warp (wid p = 0..3): NFSR b[80], feedback g and output h (34 LOP3 per
//     clock + 1 to finish z); it reads the five LFSR words a clock taps
//     (s_t for g; s_t+3, s_t+25, s_t+46, s_t+64 for h) from a shared-memory
//     ring, and writes z_t into a ring of z blocks.  Probe
//     (tools/microbench/grain_split_probe.cu): this half keeps a lone warp's
//     ALU ~94% busy.
//   L warp (wid 4 + p, same SMSP and TMEM lane quarter): LFSR s[80] (f = 3
//     LOP3 per clock), running up to 5 blocks of 32 clocks ahead of N, plus the
//     ROW_MAJOR writer of rowmajor_ws.cuh: 32x32 transposes of N's z blocks
//     into TMEM (64 B per row, wide_col) and the 64 B flushes.
//
// The LFSR sequence of an item is kept by word index i (s_{t0 + i}, t0 = the
// item's first clock): L writes its 80 entry words, then word 80 + t at its
// clock t; N's clock t reads words t, t+3, t+25, t+46, t+64.  Ring = 8 blocks
// of 32 words per lane ([block][word][lane], 32 KB per pair); word i lives in
// ring block (q0 + i/32) % 8, q0 = the pair's running block count at the item
// start.  Hand-offs are mbarriers (count 32) indexed by that running count:
//   sFull[g % 8]  L -> N : s-block g done (words up to 80 + 32(g-q0) + 31)
//   nDone[g % 8]  N -> L : N block g done (ring blocks it read are free)
//   zFull[g % 4]  N -> L : z block g written;  zEmpty[g % 4]  L -> N : read
// N block j needs words up to 32j + 95 = L's s-block j; L's s-block c
// overwrites the ring block last read by N block c - 5.
#pragma once
#include <cstdint>

#include "grain.cuh"
#include "rowmajor_ws.cuh"

namespace bsk {
namespace gsplit {

constexpr int NPAIR = 4;
constexpr int BLOCK = 2 * NPAIR * 32;
constexpr int RING_BLOCKS = 8;                     // 32-word ring blocks per lane
constexpr int RING_WORDS = RING_BLOCKS * 32 * 32;  // per pair: [block][word][lane]
constexpr int NZ = 4;                              // z blocks in flight
constexpr int ZBUF = 32 * 32;                      // [t][lane]
constexpr int PAIR_WORDS = RING_WORDS + NZ * ZBUF;
constexpr size_t SMEM_BYTES = size_t(NPAIR) * PAIR_WORDS * 4;  // 192 KB
constexpr int LEAD = RING_BLOCKS - 3;              // L's s-block c waits for N block c - LEAD
constexpr int LAG = LEAD - 1;                      // L transposes z block c - LAG after s-block c

// named barrier of pair p (N warp + L warp, 64 threads); id 0 is __syncthreads
__device__ __forceinline__ void pair_sync(uint32_t p)
{
    asm volatile("bar.sync %0, 64;" ::"r"(p + 1) : "memory");
}

__device__ __forceinline__ uint32_t lds(uint32_t saddr)
{
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(saddr));
    return v;
}
__device__ __forceinline__ void sts(uint32_t saddr, uint32_t v)
{
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(saddr), "r"(v) : "memory");
}

// ring word i of this lane: block (q0 + i / 32) % 8, word i % 32
__device__ __forceinline__ uint32_t ring_addr(uint32_t ring, uint32_t q0, uint32_t i, uint32_t lane)
{
    return ring + ((((q0 + (i >> 5)) % RING_BLOCKS) * 32 + (i & 31)) * 32 + lane) * 4;
}

}  // namespace gsplit

__global__ void __launch_bounds__(gsplit::BLOCK, 1) grain_split_rm_kernel(const __grid_constant__ KsArgs a)
{
    using namespace gsplit;
    extern __shared__ __align__(16) uint32_t gs_smem[];  // [pair][ring | z blocks]
    __shared__ uint64_t sFull[NPAIR][RING_BLOCKS], nDone[NPAIR][RING_BLOCKS];
    __shared__ uint64_t zFull[NPAIR][NZ], zEmpty[NPAIR][NZ];
    __shared__ uint32_t s_item[NPAIR];
    __shared__ uint8_t* s_row0[NPAIR][32];
    __shared__ uint32_t s_nvalid[NPAIR][32];
    __shared__ uint32_t s_tmem;

    if (threadIdx.x == 0) {
        for (int p = 0; p < NPAIR; ++p) {
            for (int k = 0; k < RING_BLOCKS; ++k) {
                ws::mbar_init(&sFull[p][k], 32);
                ws::mbar_init(&nDone[p][k], 32);
            }
            for (int k = 0; k < NZ; ++k) {
                ws::mbar_init(&zFull[p][k], 32);
                ws::mbar_init(&zEmpty[p][k], 32);
            }
        }
    }
    (void)tmem_alloc_cta(&s_tmem, true);  // 512 columns; includes __syncthreads

    const uint32_t warp = threadIdx.x >> 5;
    const uint32_t p = warp % NPAIR;
    const bool is_n = warp < NPAIR;
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t ring = static_cast<uint32_t>(__cvta_generic_to_shared(gs_smem + p * PAIR_WORDS));
    const uint32_t zring = ring + RING_WORDS * 4;
    const uint64_t total = a.units * a.nseg;
    uint32_t q0 = 0;  // running block count of this pair (identical in both warps)

    for (;;) {
        // ---- item hand-out: N takes a ticket, waits for its segment's
        // predecessor, and publishes it to L through the pair barrier
        if (is_n) {
            __syncwarp();
            if (lane == 0) {
                const uint32_t it = atomicAdd(a.ticket, 1u);
                if (it < total) {
                    const uint64_t seg = it / a.units, w = it - seg * a.units;
                    if (seg > 0)
                        while (ld_acquire(a.flags + w) < seg) __nanosleep(128);
                }
                s_item[p] = it;
            }
            __syncwarp();
        }
        pair_sync(p);
        const uint64_t item = *reinterpret_cast<volatile uint32_t*>(&s_item[p]);
        if (item >= total) break;
        const uint64_t seg = item / a.units, w = item - seg * a.units;
        const uint64_t g = w * 32u + lane;
        const uint64_t clk_begin = seg * a.seg_clocks;
        const uint64_t left = a.nclocks - clk_begin;
        const uint32_t nblk = uint32_t((left < a.seg_clocks ? left : a.seg_clocks) >> 5);

        if (is_n) {
            // ------------------------------------------------ N: NFSR + output
            uint32_t b[80];
            {
                const uint32_t* src = opaque(a.state + g);
#pragma unroll
                for (int i = 0; i < 80; ++i) b[i] = __ldcg(src + uint64_t(80 + i) * a.Gp);
            }
            // the LFSR words of the current block's 96-word window in registers:
            // v[i] = word 32j + i; the 64 words it shares with the next block
            // are renamed, only 32 are loaded per block (5 shared-memory loads
            // per clock left N short-scoreboard-bound behind their latency)
            uint32_t v[96];
#pragma unroll
            for (int i = 0; i < 64; ++i) v[i] = 0u;
#pragma unroll 1
            for (uint32_t j = 0; j < nblk; ++j) {
                const uint32_t gb = q0 + j;
                ws::mbar_wait(&sFull[p][gb % RING_BLOCKS], (gb / RING_BLOCKS) & 1u);
                if (j == 0) {
                    const uint32_t r0 = ring + ((((q0) % RING_BLOCKS) * 32) * 32 + lane) * 4;
                    const uint32_t r1 = ring + ((((q0 + 1) % RING_BLOCKS) * 32) * 32 + lane) * 4;
#pragma unroll
                    for (int i = 0; i < 32; ++i) v[i] = gsplit::lds(r0 + i * 128);
#pragma unroll
                    for (int i = 0; i < 32; ++i) v[32 + i] = gsplit::lds(r1 + i * 128);
                }
                {
                    const uint32_t r2 = ring + ((((q0 + j + 2) % RING_BLOCKS) * 32) * 32 + lane) * 4;
#pragma unroll
                    for (int i = 0; i < 32; ++i) v[64 + i] = gsplit::lds(r2 + i * 128);
                }
                if (gb >= NZ) ws::mbar_wait(&zEmpty[p][gb % NZ], ((gb / NZ) - 1) & 1u);
                const uint32_t zb = zring + ((gb % NZ) * ZBUF + lane) * 4;
                static_for<32>([&](auto uu) {
                    constexpr int u = decltype(uu)::value;
                    const uint32_t s0 = v[u], x0 = v[u + 3], x1 = v[u + 25], x2 = v[u + 46], x3 = v[u + 64];
                    const uint32_t nb = grain::g_nfsr(s0, b);
                    // h + z (grain::output with the LFSR taps passed in)
                    const uint32_t x4 = b[63];
                    const uint32_t m = lop3<grain::MUX>(x3, x0, x4);
                    const uint32_t B0 = lop3<0xE4u>(x1, x3, x4);
                    const uint32_t B1 = lop3<0x72u>(x1, x3, x4);
                    const uint32_t B = lop3<grain::MUX>(x0, B1, B0);
                    const uint32_t w1 = lop3<grain::XOR3>(b[1], b[2], b[4]);
                    const uint32_t w2 = lop3<grain::XOR3>(b[10], b[31], b[43]);
                    const uint32_t w3 = lop3<grain::XOR3>(b[56], x1, m);
                    const uint32_t ww = lop3<grain::XOR3>(w1, w2, w3);
                    gsplit::sts(zb + u * 128, lop3<grain::XAND>(ww, x2, B));
#pragma unroll
                    for (int i = 0; i < 79; ++i) b[i] = b[i + 1];
                    b[79] = nb;
                });
                ws::mbar_arrive(&nDone[p][gb % RING_BLOCKS]);
                ws::mbar_arrive(&zFull[p][gb % NZ]);
#pragma unroll
                for (int i = 0; i < 64; ++i) v[i] = v[i + 32];
            }
            uint32_t* dst = opaque(a.state + g);
#pragma unroll
            for (int i = 0; i < 80; ++i) __stcg(dst + uint64_t(80 + i) * a.Gp, b[i]);
        } else {
            // ------------------------------ L: LFSR (runs ahead) + ROW_MAJOR writer
            uint32_t s[80];
            {
                const uint32_t* src = opaque(a.state + g);
#pragma unroll
                for (int i = 0; i < 80; ++i) s[i] = __ldcg(src + uint64_t(i) * a.Gp);
            }
            // entry words 0..79 (ring blocks q0, q0+1 and half of q0+2: all
            // consumed by the previous item before the pair barrier)
#pragma unroll
            for (int i = 0; i < 80; ++i) gsplit::sts(gsplit::ring_addr(ring, q0, i, lane), s[i]);
            __syncwarp();
            const uint32_t tm = *reinterpret_cast<volatile uint32_t*>(&s_tmem) + (p << 21);
            const uint64_t b0 = clk_begin >> 5;  // call-relative index of the item's first block
            // the writer's part for z block c of this item
            auto write_block = [&](uint32_t c) {
                const uint32_t gz = q0 + c;
                ws::mbar_wait(&zFull[p][gz % NZ], (gz / NZ) & 1u);
                const uint64_t Bc = b0 + c;
                const uint32_t k = uint32_t(Bc % ws::NSLOT);
                rowmajor_transpose_smem_tmem<Grain::MSB_FIRST, 16>(
                    gs_smem + p * PAIR_WORDS + RING_WORDS + (gz % NZ) * ZBUF + lane, tm, wide_col(k));
                ws::mbar_arrive(&zEmpty[p][gz % NZ]);
                if (k == ws::NSLOT - 1 || c + 1 == nblk) {
                    const uint32_t k_lo = k - (c < k ? c : k);
                    const uint64_t col = (Bc - (k - k_lo)) * 4;
                    const uint64_t first = (w * 32u + lane) * 32u;
                    const uint32_t nvalid = first >= a.n ? 0u : uint32_t(a.n - first < 32 ? a.n - first : 32);
                    uint8_t* row0 = static_cast<uint8_t*>(a.out) + (nvalid ? first : 0) * a.row_bytes;
                    s_row0[p][lane] = row0;
                    s_nvalid[p][lane] = nvalid;
                    __syncwarp();
                    if (k_lo == 0 && k == ws::NSLOT - 1 && ((a.row_bytes | col) & 7) == 0 &&
                        a.row_bytes < (1ull << 32))
                        rowmajor_store_tmem_wide(tm, s_row0[p], s_nvalid[p], a.row_bytes, col);
                    else
                        rowmajor_store_tmem_wide_partial(tm, row0, a.row_bytes, nvalid, k_lo, k, col);
                    __syncwarp();
                }
            };
#pragma unroll 1
            for (uint32_t c = 0; c < nblk; ++c) {
                const uint32_t gb = q0 + c;
                if (c >= uint32_t(LEAD)) ws::mbar_wait(&nDone[p][(gb - LEAD) % RING_BLOCKS], ((gb - LEAD) / RING_BLOCKS) & 1u);
                // words 80 + 32c + u: ring block (c + 2 + (16 + u) / 32) of the item
                const uint32_t wa = ring + ((((q0 + c + 2) % RING_BLOCKS) * 32 + 16) * 32 + lane) * 4;
                const uint32_t wb = ring + ((((q0 + c + 3) % RING_BLOCKS) * 32) * 32 + lane) * 4;
                static_for<32>([&](auto uu) {
                    constexpr int u = decltype(uu)::value;
                    const uint32_t fs = grain::f_lfsr(s);
                    gsplit::sts(u < 16 ? wa + u * 128 : wb + (u - 16) * 128, fs);
#pragma unroll
                    for (int i = 0; i < 79; ++i) s[i] = s[i + 1];
                    s[79] = fs;
                });
                ws::mbar_arrive(&sFull[p][gb % RING_BLOCKS]);
                // the writer trails the LFSR by LAG blocks, so N never waits
                // for LFSR words while L transposes or flushes
                if (c >= uint32_t(LAG)) write_block(c - LAG);
            }
#pragma unroll 1
            for (uint32_t c = nblk > uint32_t(LAG) ? nblk - LAG : 0; c < nblk; ++c) write_block(c);
            uint32_t* dst = opaque(a.state + g);
#pragma unroll
            for (int i = 0; i < 80; ++i) __stcg(dst + uint64_t(i) * a.Gp, s[i]);
        }
        q0 += nblk;
        // both halves of the state are stored: release the unit's next segment
        pair_sync(p);
        if (is_n && seg + 1 != a.nseg) {
            __threadfence();
            __syncwarp();
            if (lane == 0) st_release(a.flags + w, uint32_t(seg + 1));
        }
    }
    tmem_dealloc_cta(*reinterpret_cast<volatile uint32_t*>(&s_tmem), true);
}

}  // namespace bsk
