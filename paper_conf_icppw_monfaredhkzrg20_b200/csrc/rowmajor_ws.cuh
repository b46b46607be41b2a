// rowmajor_ws.cuh -- warp-specialised ROW_MAJOR keystream kernel (sm_100a).
//
// PAPER.md:673-705 (sec. 4.5): each thread puts its 32-bit output word per
// clock in shared memory; filled buffers are moved to global memory with
// coalesced writes.  Here that staging is split between two warps per SMSP:
//
//   compute warp c (wid 0..3, one per SMSP): runs the register-resident clock
//     loop of the time-segmented persistent queue (keystream.cuh) and writes
//     one slice word per clock into a ring of NZ z blocks in shared memory;
//   writer warp c+4 (same SMSP, same TMEM lane quarter): for every 32-clock
//     block transposes each thread's 32x32 bit tile (PRMT + IMAD-shift/LOP3
//     butterfly) into tensor memory -- 64 B per row: all 512 columns of the
//     lane quarter, slot columns permuted by wide_col (keystream.cuh) -- and
//     every 512 clocks writes 64 B of each of the unit's 1024 rows with
//     STG.128s of 8 rows x 64 B (tcgen05.ld.16x256b read-back, L2 evict_last).
//
// The two are chained by mbarriers (full / empty per z block).  The writer's
// transposes and its flush bursts run beside the clock loop instead of inside
// it: the compute warp issues only its cipher logic plus one STS per clock,
// and the writer's ALU work fills the issue slots a lone clock-loop warp
// leaves idle.  64 B per row per flush because that is what the DRAM needs
// (profiles/r2_flush_pattern.log: 32 B per row per flush tops out at 1.4-1.8
// TB/s for this 1024-rows-per-warp pattern, 64 B reaches 2.9-3.6 TB/s), and
// one writer per lane quarter is what lets one stream own all 512 columns.
#pragma once
#include <cstdint>

#include "keystream.cuh"

namespace bsk {
namespace ws {

constexpr int NCOMP = 4;                    // compute warps per CTA (one per SMSP)
constexpr int BLOCK = 2 * NCOMP * 32;       // + one writer warp each
// z block layout of the writer-warp kernels: lane L's 32 slice words (clock t
// at word t) at L * ZP.  The clock-loop warp stores 4 clocks per STS.128 and
// the writer loads its lane's 32 words with 8 LDS.128, both bank-conflict free
// at ZP = 36 (an 8-lane store phase covers all 32 banks).  One STS.32 per
// clock ([t][lane] layout) put 4x the shared-memory instructions into the MIO
// queue the writers' flush STGs also use.
constexpr int ZP = 36;
constexpr int ZBUF = 32 * ZP;               // words in one z block: [lane][ZP]
#ifndef WS_NZ
#define WS_NZ 8
#endif
constexpr int NZ = WS_NZ;                   // z blocks in flight per pair (absorb the flush bursts)
#ifndef WS_G
#define WS_G 4
#endif
constexpr int G = WS_G;                     // z blocks per empty-barrier wait of the clock-loop warp
static_assert(G >= 1 && G <= NZ, "a wait group must fit in the ring");
constexpr int PAIR_WORDS = NZ * ZBUF;
constexpr size_t SMEM_BYTES = size_t(NCOMP) * PAIR_WORDS * 4;  // 4.5 KB per z block: 144 KB
constexpr uint32_t NSLOT = 16;              // 32-clock blocks per 64 B row piece
#ifndef WRITER_SLEEP_NS
#define WRITER_SLEEP_NS 200
#endif

// Flush-period phase of a warp-unit (rm_phase): unit u's 64 B row pieces
// start at blocks B with (B + phase(u)) % NSLOT == 0.  Without it all units
// flush in the same block: at the paper shape (2^19 instances, one clock-loop
// warp per SMSP) 512 writers then issue 32 MB of scattered row stores at once
// every 512 clocks, and the clock-loop warps' per-clock STS queue behind those
// STGs (a build without the global stores, WS_EXPERIMENT_NO_STG, ran 25%
// faster; DESIGN.md sec. 5 "ROW_MAJOR output").  Eight even phases: the wide
// flush needs 8 B aligned pieces; used when rows are not 16 B aligned anyway.
__device__ __forceinline__ uint32_t phase(int on, uint64_t unit) { return on ? 2u * uint32_t(unit & 7u) : 0u; }

// One record per work item (not per block): the clock-loop warp writes it at
// the item's start, before it arrives on the item's first z block; the writer
// derives every block's period slot and flush flag from it.  Per-block meta
// written by lane 0 (a divergent section with two dependent shared loads)
// cost the lone clock-loop warp 6.4% of its time at the paper shape (Grain,
// measured with a build that skipped those writes).  nblk == 0 terminates.
struct Item {
    uint64_t unit;  // warp-unit (32 groups)
    uint64_t b0;    // call-relative index of the item's first 32-clock block
    uint32_t nblk;  // blocks in the item
    uint32_t pad;
};
constexpr int NITEM = 16;  // records in flight per pair (> NZ + 1: the writer lags at most NZ blocks)
static_assert(NITEM > NZ + 1, "item ring");
enum : uint32_t { F_FLUSH = 1u };

// Store z words of 4 consecutive clocks (u = 4m .. 4m+3 of a block) with one
// STS.128: zz collects them, the 4th clock's call stores.
template <int UU>
__device__ __forceinline__ void put_z4(uint32_t* zl, uint32_t (&zz)[4], uint32_t v)
{
    zz[UU & 3] = v;
    if constexpr ((UU & 3) == 3) *reinterpret_cast<uint4*>(zl + (UU & ~3)) = make_uint4(zz[0], zz[1], zz[2], zz[3]);
}

__device__ __forceinline__ uint32_t smem_u32(const void* p)
{
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar)
{
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity)
{
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}

// The writer's wait for a full z block: it is the faster side and usually
// finds the block not yet full; a tight try_wait loop keeps it eligible every
// cycle and takes issue slots from the clock-loop warp on the same SMSP (ncu:
// the writer's spin branch was executed ~75x per block), so it backs off.
__device__ __forceinline__ void mbar_wait_sleepy(uint64_t* bar, uint32_t parity)
{
    uint32_t ok;
    for (;;) {
        asm volatile(
            "{\n\t.reg .pred p;\n\t"
            "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
            "selp.u32 %0, 1, 0, p;\n\t}"
            : "=r"(ok)
            : "r"(smem_u32(bar)), "r"(parity)
            : "memory");
        if (ok) break;
        __nanosleep(WRITER_SLEEP_NS);
    }
}

}  // namespace ws

template <class C, int U>
__global__ void __launch_bounds__(ws::BLOCK, 1) keystream_rm_ws_kernel(const __grid_constant__ KsArgs a)
{
    static_assert(32 % U == 0 && U % 4 == 0, "U must divide 32 (and hold whole STS.128 groups)");
    constexpr int KB = ks_block<C, U>();
    static_assert(U % KB == 0, "the loop body must hold whole schedule blocks");
    extern __shared__ __align__(16) uint32_t pair_smem[];  // [NCOMP][NZ z blocks]
    __shared__ uint64_t bar_full[ws::NCOMP][ws::NZ], bar_empty[ws::NCOMP][ws::NZ];
    __shared__ ws::Item items[ws::NCOMP][ws::NITEM];
    __shared__ uint32_t s_item[ws::NCOMP];
    __shared__ uint32_t s_nitem[ws::NCOMP];  // items started by each compute warp
    __shared__ uint8_t* s_row0[ws::NCOMP][32];                // writer: row bases of the unit's groups
    __shared__ uint32_t s_nvalid[ws::NCOMP][32];
    __shared__ uint32_t s_tmem;

    if (threadIdx.x == 0) {
        for (int c = 0; c < ws::NCOMP; ++c) s_nitem[c] = 0;
        for (int c = 0; c < ws::NCOMP; ++c)
            for (int b = 0; b < ws::NZ; ++b) {
                ws::mbar_init(&bar_full[c][b], 32);
                ws::mbar_init(&bar_empty[c][b], 32);
            }
    }
    // all 512 columns: the writer of lane quarter p owns them for its stream
    (void)tmem_alloc_cta(&s_tmem, true);  // includes __syncthreads

    const uint32_t warp = threadIdx.x >> 5;
    const uint32_t pair = warp % ws::NCOMP;
    uint32_t* zbase = pair_smem + pair * ws::PAIR_WORDS;
    const uint64_t total = a.units * a.nseg;

    if (warp < ws::NCOMP) {
        // ------------------------------------------------------------ compute
        volatile uint32_t* slot = s_item + pair;
        next_item(a, slot);
        uint32_t seq = 0;  // z blocks handed to the writer so far
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

            if (lane == 0) {
                const uint32_t ni = s_nitem[pair];
                ws::Item& it = items[pair][ni % ws::NITEM];
                it.unit = w;
                it.b0 = clk_begin >> 5;
                it.nblk = nblk;
                s_nitem[pair] = ni + 1;
            }
            C c;
            c.load(a.state, a.Gp, g);
            // hand block blk of the item (ring slot sq) to the writer.  The
            // per-block code re-derives this warp's pair index (warp_volatile)
            // instead of keeping ring / barrier addresses live across the clock
            // loop (ptxas spilled them: an LDL on every block's critical path)
            // ring slot of z block sq (its empty barrier already waited for)
            auto slot_ptr = [&](uint32_t sq) {
                const uint32_t pv = warp_volatile(), b = sq % ws::NZ;
                return pair_smem + pv * ws::PAIR_WORDS + b * ws::ZBUF + laneid_volatile() * ws::ZP;
            };
            // The writer consumes z blocks in order, so slot sq's empty barrier
            // having completed its phase implies the same for every earlier
            // slot: one wait covers a group of WS_G blocks (the try_wait's
            // round trip stalled the lone clock-loop warp once per block).
            auto wait_empty = [&](uint32_t sq) {
                if (sq >= ws::NZ) {
                    const uint32_t pv = warp_volatile(), b = sq % ws::NZ;
                    ws::mbar_wait(&bar_empty[pv][b], ((sq / ws::NZ) - 1) & 1u);
                }
            };
            auto acquire = [&](uint32_t sq) {
                wait_empty(sq);
                return slot_ptr(sq);
            };
            // z block sq complete (the writer derives its slot from the item record)
            auto publish = [&](uint32_t sq, uint32_t) {
                const uint32_t pv = warp_volatile(), b = sq % ws::NZ;
                ws::mbar_arrive(&bar_full[pv][b]);
            };
            uint32_t blk = 0;
            if constexpr (ks_period<C>::value) {
                // whole rotation periods without register moves (Lfsr128:
                // 4.0 instead of 8.5 instructions per clock, C2 26.4 vs 25.3 Tb/s)
                constexpr int PB = C::PERIOD_BLOCKS;
#pragma unroll 1
                for (; blk + PB <= nblk; blk += PB, seq += PB) {
                    static_for<PB>([&](auto jj) {
                        constexpr int J = decltype(jj)::value;
                        uint32_t* zb = acquire(seq + J);
                        uint32_t zz[4];
                        c.template period_block<J>([&](auto u, uint32_t v) { ws::put_z4<decltype(u)::value>(zb, zz, v); });
                        publish(seq + J, blk + J);
                    });
                }
            }
#pragma unroll 1
            while (blk < nblk) {
                const uint32_t gn = nblk - blk < uint32_t(ws::G) ? nblk - blk : uint32_t(ws::G);
                wait_empty(seq + gn - 1);
#pragma unroll 1
                for (uint32_t gi = 0; gi < gn; ++gi, ++blk, ++seq) {
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
        const uint32_t b = seq % ws::NZ;
        if (seq >= ws::NZ) ws::mbar_wait(&bar_empty[pair][b], ((seq / ws::NZ) - 1) & 1u);
        if (laneid_volatile() == 0) items[pair][s_nitem[pair] % ws::NITEM].nblk = 0;  // terminate record
        ws::mbar_arrive(&bar_full[pair][b]);
    } else {
        // ------------------------------------------------------------- writer
        const uint32_t lane = threadIdx.x & 31u;
        uint64_t unit = 0, b0 = 0;
        uint32_t nblk = 0, seq0 = 0, nrec = 0;
        for (uint32_t seq = 0;; ++seq) {
            const uint32_t b = seq % ws::NZ;
            ws::mbar_wait_sleepy(&bar_full[pair][b], (seq / ws::NZ) & 1u);
            if (seq == seq0 + nblk) {  // the next item's first block (or the terminate marker)
                const volatile ws::Item& it = items[pair][nrec % ws::NITEM];
                ++nrec;
                nblk = it.nblk;
                if (nblk == 0) break;
                unit = it.unit;
                b0 = it.b0;
                seq0 = seq;
            }
            const uint32_t blk = seq - seq0;
            const uint64_t B = b0 + blk;
            const uint32_t k = uint32_t((B + ws::phase(a.rm_phase, unit)) % ws::NSLOT);
            const uint32_t k_lo = k - (blk < k ? blk : k);
            const uint32_t flags = (k == ws::NSLOT - 1 || blk + 1 == nblk) ? ws::F_FLUSH : 0u;
            const uint32_t tm = *reinterpret_cast<volatile uint32_t*>(&s_tmem) + (pair << 21);
            // WS_EXPERIMENT_NO_WRITER (measurement builds only, wrong output):
            // the writer skips its transposes and flushes, which isolates the
            // lone clock-loop warp's own rate
#ifndef WS_EXPERIMENT_NO_WRITER
            rowmajor_transpose_lanes_tmem<C::MSB_FIRST, 16>(zbase + b * ws::ZBUF + lane * ws::ZP, tm, wide_col(k));
#endif
            ws::mbar_arrive(&bar_empty[pair][b]);
#if defined(WS_EXPERIMENT_NO_WRITER) || defined(WS_EXPERIMENT_NO_FLUSH)
            if (false) {
#else
            if (flags & ws::F_FLUSH) {
#endif
                const uint64_t first = (unit * 32u + lane) * 32u;
                const uint32_t nvalid = first >= a.n ? 0u : uint32_t(a.n - first < 32 ? a.n - first : 32);
                uint8_t* row0 = static_cast<uint8_t*>(a.out) + (nvalid ? first : 0) * a.row_bytes;
                const uint64_t col = (B - (k - k_lo)) * 4;
                s_row0[pair][lane] = row0;
                s_nvalid[pair][lane] = nvalid;
                __syncwarp();
                if (k_lo == 0 && k == ws::NSLOT - 1 && ((a.row_bytes | col) & 7) == 0 && a.row_bytes < (1ull << 32))
                    rowmajor_store_tmem_wide(tm, s_row0[pair], s_nvalid[pair], a.row_bytes, col);
                else
                    rowmajor_store_tmem_wide_partial(tm, s_row0[pair], s_nvalid[pair], a.row_bytes, k_lo, k, col);
                __syncwarp();
            }
        }
    }
    tmem_dealloc_cta(*reinterpret_cast<volatile uint32_t*>(&s_tmem), true);
}

}  // namespace bsk
