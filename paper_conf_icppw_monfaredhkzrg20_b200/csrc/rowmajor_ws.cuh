// rowmajor_ws.cuh -- warp-specialised ROW_MAJOR keystream kernel (sm_100a).
//
// PAPER.md:673-705 (sec. 4.5): each thread puts its 32-bit output word per
// clock in shared memory; filled buffers are moved to global memory with
// coalesced writes.  Here that staging is split between two warps per SMSP:
//
//   compute warp c (wid 0..3, one per SMSP): runs the register-resident clock
//     loop of the time-segmented persistent queue (keystream.cuh) and writes
//     one slice word per clock into a double-buffered z block in smem;
//   writer warp c+4 (same SMSP): for every 32-clock block transposes each
//     thread's 32x32 bit tile (PRMT + IMAD-shift/LOP3 butterfly), parks the
//     row words in a 32 B-sector buffer and every 256 clocks writes whole
//     sectors of every instance row (two 16 B stores per row).
//
// The two are chained by mbarriers (full / empty per z buffer).  The writer's
// shared-memory and store latencies hide behind the compute warp's LOP3
// stream instead of stalling it, and the writer's transpose work fills ALU
// issue slots the compute warp leaves idle.
#pragma once
#include <cstdint>

#include "keystream.cuh"

namespace bsk {
namespace ws {

constexpr int NCOMP = 4;                    // compute warps per CTA (one per SMSP)
constexpr int BLOCK = 2 * NCOMP * 32;       // + one writer warp each
constexpr int ZBUF = 32 * 32;               // words in one z block: [t][lane]
constexpr int PAIR_WORDS = 2 * ZBUF + OS_WORDS;
constexpr size_t SMEM_BYTES = size_t(NCOMP) * PAIR_WORDS * 4;  // 160 KB

struct Meta {
    uint64_t unit;   // warp-unit of the item (32 groups)
    uint64_t B;      // call-relative index of this 32-clock block
    uint32_t k_lo;   // first staged sector slot to write on flush
    uint32_t flags;  // F_FLUSH | F_TERM
};
enum : uint32_t { F_FLUSH = 1u, F_TERM = 2u };

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

}  // namespace ws

template <class C, int U>
__global__ void __launch_bounds__(ws::BLOCK, 1) keystream_rm_ws_kernel(const __grid_constant__ KsArgs a)
{
    static_assert(32 % U == 0, "U must divide 32");
    constexpr int KB = ks_block<C, U>();
    static_assert(U % KB == 0, "the loop body must hold whole schedule blocks");
    extern __shared__ uint32_t pair_smem[];  // [NCOMP][2 z blocks + sector buffer]
    __shared__ uint64_t bar_full[ws::NCOMP][2], bar_empty[ws::NCOMP][2];
    __shared__ ws::Meta meta[ws::NCOMP][2];
    __shared__ uint32_t s_item[ws::NCOMP];
    __shared__ uint64_t s_unit[ws::NCOMP], s_b0[ws::NCOMP];  // per-item context of each compute warp

    if (threadIdx.x == 0) {
        for (int c = 0; c < ws::NCOMP; ++c)
            for (int b = 0; b < 2; ++b) {
                ws::mbar_init(&bar_full[c][b], 32);
                ws::mbar_init(&bar_empty[c][b], 32);
            }
    }
    __syncthreads();

    const uint32_t warp = threadIdx.x >> 5;
    const uint32_t pair = warp % ws::NCOMP;
    uint32_t* zbase = pair_smem + pair * ws::PAIR_WORDS;
    uint32_t* os = zbase + 2 * ws::ZBUF;
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
                s_unit[pair] = w;
                s_b0[pair] = clk_begin >> 5;
            }
            C c;
            c.load(a.state, a.Gp, g);
#pragma unroll 1
            for (uint32_t blk = 0; blk < nblk; ++blk, ++seq) {
                const uint32_t b = seq & 1u;
                if (seq >= 2) ws::mbar_wait(&bar_empty[pair][b], ((seq >> 1) - 1) & 1u);
                uint32_t* zb = zbase + b * ws::ZBUF + laneid_volatile();
#pragma unroll 1
                for (uint32_t k = 0; k < 32; k += U) {
                    static_for<U>([&](auto u) {
                        constexpr int J = decltype(u)::value % KB;
                        zb[(k + decltype(u)::value) * 32] = ks_z<J, KB>(c);
                        ks_clock<J, KB>(c);
                    });
                }
                if (laneid_volatile() == 0) {
                    const uint64_t B = s_b0[pair] + blk;
                    const uint32_t kk = uint32_t(B & 7);
                    ws::Meta& m = meta[pair][b];
                    m.unit = s_unit[pair];
                    m.B = B;
                    m.k_lo = kk - (blk < kk ? blk : kk);
                    m.flags = (kk == 7 || blk + 1 == nblk) ? ws::F_FLUSH : 0u;
                }
                ws::mbar_arrive(&bar_full[pair][b]);
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
        const uint32_t b = seq & 1u;
        if (seq >= 2) ws::mbar_wait(&bar_empty[pair][b], ((seq >> 1) - 1) & 1u);
        if (laneid_volatile() == 0) meta[pair][b].flags = ws::F_TERM;
        ws::mbar_arrive(&bar_full[pair][b]);
    } else {
        // ------------------------------------------------------------- writer
        const uint32_t lane = threadIdx.x & 31u;
        for (uint32_t seq = 0;; ++seq) {
            const uint32_t b = seq & 1u;
            ws::mbar_wait(&bar_full[pair][b], (seq >> 1) & 1u);
            const volatile ws::Meta& vm = meta[pair][b];
            const uint32_t flags = vm.flags;
            if (flags & ws::F_TERM) break;
            const uint64_t unit = vm.unit, B = vm.B;
            const uint32_t k_lo = vm.k_lo;
            const uint32_t k = uint32_t(B & 7);
            rowmajor_transpose<C::MSB_FIRST>(zbase + b * ws::ZBUF + lane, os + lane, k);
            ws::mbar_arrive(&bar_empty[pair][b]);
            if (flags & ws::F_FLUSH) {
                const uint64_t first = (unit * 32u + lane) * 32u;
                const uint32_t nvalid = first >= a.n ? 0u : uint32_t(a.n - first < 32 ? a.n - first : 32);
                uint8_t* row0 = static_cast<uint8_t*>(a.out) + (nvalid ? first : 0) * a.row_bytes;
                rowmajor_store(os + lane, row0, a.row_bytes, nvalid, k_lo, k, (B - (k - k_lo)) * 4);
            }
        }
    }
}

}  // namespace bsk
