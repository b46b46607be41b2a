// rowmajor_ws2.cuh -- ROW_MAJOR keystream kernel with two writer warps per
// clock-loop warp and 128 B per row per flush (sm_100a), for ciphers whose
// clock logic is cheap enough that the output path is the whole cost (the
// paper's bitsliced LFSR, sec. 4.3).
//
// PAPER.md:673-705 (sec. 4.5): the output words of each clock are staged and
// moved to global memory with coalesced writes.  What the DRAM needs from a
// 1024-rows-per-stream output (tools/microbench/flush_pattern.cu,
// profiles/r2_flush_pattern.log): rowmajor_ws.cuh's 4 streams per SM with 64 B
// per row per flush reach 3.5 TB/s; 2 streams per SM (half the rows in flight)
// with 128 B per row per flush, each row's 128 B written as two halves by two
// warps, reach 4.65 TB/s.  Here:
//
//   clock-loop warp 4 + s (s = 0, 1; one per stream): the register-resident
//     clock loop of the time-segmented persistent queue, one slice word per
//     clock into a ring of NZ = 16 z blocks of its stream;
//   writer warps 2s, 2s + 1 (TMEM lane quarters 2s, 2s + 1): a 128 B row
//     piece is a period of 32 blocks (period slot k = block B mod 32, 4 B of
//     each row); writer w owns the slots with bit 3 of k equal to w, i.e. the
//     32 B sectors w and 2 + w of the piece.  It transposes each of its blocks
//     into its quarter (local slot k' = 8 (k >> 4) + (k & 7): 16 slots = 64 B
//     per row, all 512 columns, wide_col permutation) and flushes its two
//     sectors of every row when its last block of the period is in; the
//     other writer's flush of the same lines follows within a few blocks, so
//     L2 (evict_last) sees whole 128 B lines.
//
// A writer takes its blocks in pairs (one full-barrier wait per pair) and
// transposes two consecutive blocks of one item together (F_PAIR), writing
// each row's two words with one tcgen05.st.32x32b.x2: twice the independent
// work for a latency-bound lone warp (LFSR C2 27.3 -> 28.7 Tb/s).
//
// Ring sequence: block seq sits in ring slot seq % 16 and belongs to writer
// (seq >> 3) & 1, so each writer walks its own 8 slots; the clock-loop warp
// keeps seq = B (mod 16) by publishing skip blocks at item starts, which
// makes the sequence owner the period-slot owner.  Both writers get a
// terminate block at the end.
#pragma once
#include <cstdint>

#include "keystream.cuh"
#include "rowmajor_ws.cuh"

namespace bsk {
namespace ws2 {

constexpr int NSTREAM = 2;                      // clock-loop warps per CTA (warps 4, 5)
constexpr int NWRITER = 4;                      // writer warps 0..3 (lane quarter = warp index)
constexpr int BLOCK = (NWRITER + NSTREAM) * 32;
constexpr int ZBUF = ws::ZBUF;                  // words in one z block: [lane][ws::ZP]
#ifndef WS2_NZ
#define WS2_NZ 16
#endif
// ring slots per stream (multiple of 8): block seq -> slot seq % NZ, owner (seq >> 3) & 1
constexpr int NZ = WS2_NZ;
static_assert(NZ % 8 == 0 && NZ >= 16, "whole 8-block owner groups, at least one per writer");
constexpr size_t SMEM_BYTES = size_t(NSTREAM) * NZ * ZBUF * 4;  // 144 KB at NZ = 16
constexpr uint32_t PERIOD = 32;                 // 32-clock blocks per 128 B row piece

struct Meta {
    uint64_t unit;
    uint64_t B;      // call-relative block index
    uint32_t k_lo;   // first period slot of the item in this period
    uint32_t flags;  // F_FLUSH | F_TERM | F_SKIP
};
// F_PAIR: an even block whose successor is the same item's next block (the
// writer transposes the two together)
enum : uint32_t { F_FLUSH = 1u, F_TERM = 2u, F_SKIP = 4u, F_PAIR = 8u };

#ifndef WS2_BACKOFF_NS
#define WS2_BACKOFF_NS 64
#endif
// try_wait with a short back-off once the first probe fails
__device__ __forceinline__ void mbar_wait_backoff(uint64_t* bar, uint32_t parity)
{
    uint32_t ok;
    for (;;) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(ws::smem_u32(bar)), "r"(parity)
            : "memory");
        if (ok) break;
        __nanosleep(WS2_BACKOFF_NS);
    }
}

// period slot of thread j's first slot (of 4) in writer w's flush read-back
__device__ __forceinline__ uint32_t thread_slot0(uint32_t j, uint32_t w)
{
    return 16 * (j >> 1) + 8 * w + 4 * (j & 1);
}

// Flush writer w's sectors of slots [k_lo, k_hi] (period slots) of every real
// row from its TMEM quarter.  col = byte offset of slot k_lo in the rows.
// 16x256b.x8 read-back: thread j = t % 4 holds local slots 4j..4j+3 (16 B) of
// rows q..q+3 of lanes la, lb; whole periods with 16 B aligned rows store one
// STG.128 per thread and row, anything else the widest aligned pieces.
__device__ __forceinline__ void store_split(uint32_t tm, uint8_t* const* row0s, const uint32_t* nvalids,
                                            uint64_t row_bytes, uint32_t w, uint32_t k_lo, uint32_t k_hi, uint64_t col)
{
    tmem_wait_st();
    const uint32_t t = laneid_volatile();
    const uint32_t j = t & 3u;
    const uint64_t pol = l2_evict_last_policy();
    const uint32_t ps0 = thread_slot0(j, w);
    // every slot of the writer's two sectors present: k_hi = its last slot (23 or 31)
    const bool whole = k_lo == 0 && k_hi == (w ? 31u : 23u) && ((row_bytes | col) & 15) == 0;
    const int lo = int(k_lo > ps0 ? k_lo : ps0), hi = int(k_hi < ps0 + 3 ? k_hi : ps0 + 3);
    const int m0 = lo - int(ps0), m1 = hi - int(ps0);
    const int64_t off = int64_t(col) + 4 * (int64_t(ps0) - int64_t(k_lo));
#pragma unroll 1
    for (uint32_t h = 0; h < 2; ++h) {
        const uint32_t la = 16 * h + (t >> 2), lb = la + 8;
        uint8_t* pa = row0s[la] + off;
        uint8_t* pb = row0s[lb] + off;
        const uint32_t na = nvalids[la], nb = nvalids[lb];
        if (whole && __all_sync(0xFFFFFFFFu, (na & nb) == 32)) {
#pragma unroll 1
            for (uint32_t q = 0; q < 32; q += 4) {
                uint32_t v[32];
                tmem_ld16x256b_x8(tm + ((16 * h) << 16) + q * 16, v);
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    st128_hint(pa, v[8 * r], v[8 * r + 1], v[8 * r + 4], v[8 * r + 5], pol);
                    st128_hint(pb, v[8 * r + 2], v[8 * r + 3], v[8 * r + 6], v[8 * r + 7], pol);
                    pa = add_fma(pa, row_bytes);
                    pb = add_fma(pb, row_bytes);
                }
            }
            continue;
        }
#pragma unroll 1
        for (uint32_t q = 0; q < 32; q += 4) {
            uint32_t v[32];
            tmem_ld16x256b_x8(tm + ((16 * h) << 16) + q * 16, v);
            if (m0 <= m1) {
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    if (q + r < na) st_run4(pa, v[8 * r], v[8 * r + 1], v[8 * r + 4], v[8 * r + 5], m0, m1, pol);
                    if (q + r < nb) st_run4(pb, v[8 * r + 2], v[8 * r + 3], v[8 * r + 6], v[8 * r + 7], m0, m1, pol);
                    pa += row_bytes;
                    pb += row_bytes;
                }
            }
        }
    }
}

}  // namespace ws2

template <class C, int U>
__global__ void __launch_bounds__(ws2::BLOCK, 1) keystream_rm_ws2_kernel(const __grid_constant__ KsArgs a)
{
    static_assert(32 % U == 0, "U must divide 32");
    constexpr int KB = ks_block<C, U>();
    static_assert(U % KB == 0, "the loop body must hold whole schedule blocks");
    extern __shared__ __align__(1024) uint32_t ring_smem[];  // [NSTREAM][NZ z blocks]
    __shared__ uint64_t bar_full[ws2::NSTREAM][ws2::NZ], bar_empty[ws2::NSTREAM][ws2::NZ];
    __shared__ ws2::Meta meta[ws2::NSTREAM][ws2::NZ];
    __shared__ uint32_t s_item[ws2::NSTREAM];
    __shared__ uint64_t s_unit[ws2::NSTREAM], s_b0[ws2::NSTREAM];
    __shared__ uint8_t* s_row0[ws2::NWRITER][32];
    __shared__ uint32_t s_nvalid[ws2::NWRITER][32];
    __shared__ uint32_t s_tmem;

    if (threadIdx.x == 0) {
        for (int s = 0; s < ws2::NSTREAM; ++s)
            for (int b = 0; b < ws2::NZ; ++b) {
                ws::mbar_init(&bar_full[s][b], 32);
                ws::mbar_init(&bar_empty[s][b], 32);
            }
    }
    (void)tmem_alloc_cta(&s_tmem, true);  // all 512 columns; includes __syncthreads

    const uint32_t warp = threadIdx.x >> 5;
    const uint64_t total = a.units * a.nseg;

    if (warp >= ws2::NWRITER) {
        // ------------------------------------------------------------ compute
        const uint32_t sid = warp - ws2::NWRITER;
        volatile uint32_t* slot = s_item + sid;
        // ring / barrier addresses are re-derived per block from the warp index
        // (kept out of the register-saturated clock loop, rowmajor_ws.cuh)
        auto sidv = [&]() { return warp_volatile() - uint32_t(ws2::NWRITER); };
        auto slot_ptr = [&](uint32_t sq) {
            return ring_smem + (sidv() * ws2::NZ + sq % ws2::NZ) * ws2::ZBUF + laneid_volatile() * ws::ZP;
        };
        // (backs off while waiting: the writer it waits for may share its SMSP)
        auto wait_empty = [&](uint32_t sq) {
            if (sq >= uint32_t(ws2::NZ))
                ws2::mbar_wait_backoff(&bar_empty[sidv()][sq % ws2::NZ], ((sq / ws2::NZ) - 1) & 1u);
        };
        // meta of block sq + arrive on its full barrier (lane 0 writes meta)
        auto post = [&](uint32_t sq, uint64_t unit, uint64_t B, uint32_t k_lo, uint32_t flags) {
            const uint32_t sv = sidv(), b = sq % ws2::NZ;
            if (laneid_volatile() == 0) {
                ws2::Meta& m = meta[sv][b];
                m.unit = unit;
                m.B = B;
                m.k_lo = k_lo;
                m.flags = flags;
            }
            ws::mbar_arrive(&bar_full[sv][b]);
        };
        next_item(a, slot);
        uint32_t seq = 0;
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
            const uint32_t nblk = uint32_t((left < a.seg_clocks ? left : a.seg_clocks) >> 5);
            const uint32_t B0 = uint32_t(clk_begin >> 5);
            // skip blocks until seq = B0 (mod 16): sequence owner = period-slot owner
            while ((seq - B0) & 15u) {
                wait_empty(seq);
                post(seq, 0, 0, 0, ws2::F_SKIP);
                ++seq;
            }
            if (lane == 0) {
                s_unit[sid] = w;
                s_b0[sid] = clk_begin >> 5;
            }
            C c;
            c.load(a.state, a.Gp, g);
            auto publish = [&](uint32_t sq, uint32_t blk) {
                const uint32_t sv = sidv(), b = sq % ws2::NZ;
                if (laneid_volatile() == 0) {
                    const uint64_t B = s_b0[sv] + blk;
                    const uint32_t k = uint32_t(B % ws2::PERIOD);
                    // flush when the owner has no later block in this period and item
                    const uint32_t nk = (k & 7u) != 7u ? k + 1 : k + 9;
                    const bool fl = nk >= ws2::PERIOD || blk + (nk - k) >= nblk;
                    ws2::Meta& m = meta[sv][b];
                    m.unit = s_unit[sv];
                    m.B = B;
                    m.k_lo = k - (blk < k ? blk : k);
                    m.flags = (fl ? ws2::F_FLUSH : 0u) | ((B & 1u) == 0 && blk + 1 < nblk ? ws2::F_PAIR : 0u);
                }
                ws::mbar_arrive(&bar_full[sv][b]);
            };
            uint32_t blk = 0;
            if constexpr (ks_period<C>::value) {
                constexpr int PB = C::PERIOD_BLOCKS;
                static_assert(PB == 4, "one empty wait per 4 blocks of one owner");
#pragma unroll 1
                for (; blk + PB <= nblk; blk += PB, seq += PB) {
                    const bool grouped = (seq & 3u) == 0;
                    if (grouped) wait_empty(seq + PB - 1);
                    static_for<PB>([&](auto jj) {
                        constexpr int J = decltype(jj)::value;
                        if (!grouped) wait_empty(seq + J);
                        uint32_t* zb = slot_ptr(seq + J);
                        uint32_t zz[4];
                        c.template period_block<J>([&](auto u, uint32_t v) { ws::put_z4<decltype(u)::value>(zb, zz, v); });
                        publish(seq + J, blk + J);
                    });
                }
            }
#pragma unroll 1
            for (; blk < nblk; ++blk, ++seq) {
                wait_empty(seq);
                uint32_t* zb = slot_ptr(seq);
#pragma unroll 1
                for (uint32_t k = 0; k < 32; k += U) {
                    uint32_t zz[4];
                    static_for<U>([&](auto u) {
                        constexpr int J = decltype(u)::value % KB;
                        ws::put_z4<decltype(u)::value>(zb + k, zz, ks_z<J, KB>(c));
                        ks_clock<J, KB>(c);
                    });
                }
                publish(seq, blk);
            }
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
        // terminate both writers: writer 0 at the next seq = 0 (mod 16),
        // writer 1 eight blocks later (its next slot)
        while (seq & 15u) {
            wait_empty(seq);
            post(seq, 0, 0, 0, ws2::F_SKIP);
            ++seq;
        }
        // (writers take their blocks in pairs: terminate both blocks of each pair)
        for (uint32_t e : {0u, 1u, 8u, 9u}) {
            wait_empty(seq + e);
            post(seq + e, 0, 0, 0, ws2::F_TERM);
        }
    } else {
        // ------------------------------------------------------------- writer
        const uint32_t sid = warp >> 1, wr = warp & 1u;
        const uint32_t lane = threadIdx.x & 31u;
        uint32_t* zbase = ring_smem + sid * ws2::NZ * ws2::ZBUF;
        // Blocks are taken in pairs (i, i + 1 of the writer's 8-block groups):
        // one full-barrier wait per pair, on the second block -- the clock-loop
        // warp arrives on the pair's barriers in order, so the second one's
        // phase completing implies the first one's.  The try_wait's latency
        // (~90 cycles even when complete) and the wait loop's branch
        // resolution were ~20% of the writers' stall samples at one per block.
        for (uint32_t i = 0;; ++i) {
            // this writer's i-th block: sequence number, ring slot, slot use count
            const uint32_t sq = 16 * (i >> 3) + 8 * wr + (i & 7u);
            const uint32_t b = sq % ws2::NZ;
            if ((i & 1u) == 0)
                ws::mbar_wait_sleepy(&bar_full[sid][(sq + 1) % ws2::NZ], ((sq + 1) / ws2::NZ) & 1u);
            const volatile ws2::Meta& vm = meta[sid][b];
            const uint32_t flags = vm.flags;
            if (flags & ws2::F_TERM) break;
            // Both blocks of a pair consecutive blocks of one item (F_PAIR): they
            // sit at consecutive local slots (seq = B (mod 16), B even, kl even)
            // and the first one does not end the writer's period (only an item's
            // last block would).  One paired transpose.
            if ((i & 1u) == 0 && (flags & ws2::F_PAIR)) {
                const uint32_t b1 = (sq + 1) % ws2::NZ;
                const volatile ws2::Meta& vm1 = meta[sid][b1];
                const uint32_t flags1 = vm1.flags;
                {
                    const uint64_t unit = vm1.unit, B = vm1.B;
                    const uint32_t k_lo = vm1.k_lo;
                    const uint32_t k = uint32_t(B % ws2::PERIOD);
                    const uint32_t kl = 8 * (k >> 4) + (k & 7u) - 1;  // the pair's first (even) local slot
                    const uint32_t tm = *reinterpret_cast<volatile uint32_t*>(&s_tmem) + (warp << 21);
                    rowmajor_transpose_lanes_tmem2<C::MSB_FIRST, 16>(zbase + b * ws2::ZBUF + lane * ws::ZP,
                                                                     zbase + b1 * ws2::ZBUF + lane * ws::ZP, tm,
                                                                     wide_col(kl));
                    ws::mbar_arrive(&bar_empty[sid][b]);
                    ws::mbar_arrive(&bar_empty[sid][b1]);
                    ++i;  // the pair's second block is done as well
                    if (flags1 & ws2::F_FLUSH) {
                        const uint64_t first = (unit * 32u + lane) * 32u;
                        const uint32_t nvalid = first >= a.n ? 0u : uint32_t(a.n - first < 32 ? a.n - first : 32);
                        s_row0[warp][lane] = static_cast<uint8_t*>(a.out) + (nvalid ? first : 0) * a.row_bytes;
                        s_nvalid[warp][lane] = nvalid;
                        __syncwarp();
                        const uint64_t col = (B - (k - k_lo)) * 4;
                        ws2::store_split(tm, s_row0[warp], s_nvalid[warp], a.row_bytes, wr, k_lo, k, col);
                        __syncwarp();
                    }
                    continue;
                }
            }
            if (flags & ws2::F_SKIP) {
                ws::mbar_arrive(&bar_empty[sid][b]);
                continue;
            }
            const uint64_t unit = vm.unit, B = vm.B;
            const uint32_t k_lo = vm.k_lo;
            const uint32_t k = uint32_t(B % ws2::PERIOD);
            const uint32_t kl = 8 * (k >> 4) + (k & 7u);  // local slot in this writer's quarter
            const uint32_t tm = *reinterpret_cast<volatile uint32_t*>(&s_tmem) + (warp << 21);
            rowmajor_transpose_lanes_tmem<C::MSB_FIRST, 16>(zbase + b * ws2::ZBUF + lane * ws::ZP, tm, wide_col(kl));
            ws::mbar_arrive(&bar_empty[sid][b]);
            if (flags & ws2::F_FLUSH) {
                const uint64_t first = (unit * 32u + lane) * 32u;
                const uint32_t nvalid = first >= a.n ? 0u : uint32_t(a.n - first < 32 ? a.n - first : 32);
                s_row0[warp][lane] = static_cast<uint8_t*>(a.out) + (nvalid ? first : 0) * a.row_bytes;
                s_nvalid[warp][lane] = nvalid;
                __syncwarp();
                const uint64_t col = (B - (k - k_lo)) * 4;
                ws2::store_split(tm, s_row0[warp], s_nvalid[warp], a.row_bytes, wr, k_lo, k, col);
                __syncwarp();
            }
        }
    }
    tmem_dealloc_cta(*reinterpret_cast<volatile uint32_t*>(&s_tmem), true);
}

}  // namespace bsk
