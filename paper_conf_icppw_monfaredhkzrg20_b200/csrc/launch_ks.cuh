// launch_ks.cuh -- host launcher of the stream-cipher keystream kernel
// (keystream.cuh / rowmajor_ws.cuh), included by the per-cipher translation
// units cipher_mickey2.cu, cipher_grain.cu and cipher_lfsr.cu.
//
// Kernel instances built per cipher C (the only ones the options can reach):
//   CHECKSUM, SLICED      : keystream_kernel<C, L, U>                 U in {U_DEFAULT, U_ALT0, U_ALT1}
//   ROW_MAJOR, smem       : keystream_kernel<C, ROW_MAJOR, U>         (8 sector slots, z block in regs at U = 32)
//   ROW_MAJOR, TMEM       : keystream_kernel<C, ROW_MAJOR, U, .., TMEM>
//   ROW_MAJOR, TMEM + dbl : keystream_kernel<C, ROW_MAJOR, U, .., TMEM, DBL>
//   ROW_MAJOR, TMEM 64 B  : keystream_kernel<C, ROW_MAJOR, U, .., TMEM, -, WIDE>
//   ROW_MAJOR, specialised: keystream_rm_ws_kernel<C, U>   (compute + writer warps, TMEM 64 B staging)
//   ROW_MAJOR, 2 writers  : keystream_rm_ws2_kernel<C, U>  (per clock-loop warp; 128 B per row per flush)
#pragma once
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "internal.h"
#include "keystream.cuh"
#include "rowmajor_ws.cuh"
#include "rowmajor_ws2.cuh"

namespace bsrng_impl {

constexpr int KS_BLOCK = 128;

template <class C, int LAYOUT, bool TMEM = false, bool DBL = false, bool WIDE = false>
auto pick_keystream_kernel(const bsrng_t* h, int* U)
{
    auto kern = &bsk::keystream_kernel<C, LAYOUT, C::U_DEFAULT, KS_BLOCK, 8, true, TMEM, DBL, WIDE>;
    *U = C::U_DEFAULT;
    if (h->opt_unroll == C::U_ALT0)
        kern = &bsk::keystream_kernel<C, LAYOUT, C::U_ALT0, KS_BLOCK, 8, true, TMEM, DBL, WIDE>, *U = C::U_ALT0;
    if (h->opt_unroll == C::U_ALT1)
        kern = &bsk::keystream_kernel<C, LAYOUT, C::U_ALT1, KS_BLOCK, 8, true, TMEM, DBL, WIDE>, *U = C::U_ALT1;
    return kern;
}

template <class C, int LAYOUT>
int launch_keystream(bsrng_t* h, void* out, uint64_t bits, cudaStream_t st)
{
    constexpr bool RM = LAYOUT == bsk::L_ROW_MAJOR;
    // ROW_MAJOR kernel: warp-specialised compute/writer kernel (rowmajor_ws.cuh,
    // 8 warps per CTA of which 4 run the clock loop; always persistent), or
    // the plain clock kernel with the row segments staged in tensor memory
    // (TMEM) or shared memory.  Defaults per cipher (RM_TMEM traits).
    // auto (C::RM_WS): 0 never, 1 when every warp-unit gets its own SMSP
    // (lone clock-loop warps), 2 always
    const bool lone = h->units <= uint64_t(h->num_sms) * 4;
    // (an explicit plain-kernel staging choice -- rm_wide, rm_tmem -- turns the
    // automatic writer-warp choice off)
    const bool plain_asked = h->opt_rm_wide > 0 || h->opt_rm_tmem >= 0;
    // 3: the two-writers-per-stream kernel (rowmajor_ws2.cuh, 128 B per row per flush)
    const int ws_kind = h->opt_rm_ws < 0
                            ? (plain_asked ? 0 : C::RM_WS == 3 ? 2 : (C::RM_WS == 2 || (C::RM_WS == 1 && lone)) ? 1 : 0)
                            : h->opt_rm_ws;
    // calls longer than MAX_SEG_CLOCKS need time segments, i.e. the persistent queue
    const bool persistent = h->opt_sched != 0 || bits > MAX_SEG_CLOCKS;
    const bool ws2 = RM && ws_kind == 2 && persistent;
    const bool ws = RM && ws_kind != 0 && persistent;
    // 64 B TMEM staging (keystream.cuh wide_col): one clock-loop warp per
    // SMSP with all 512 columns, so each flush writes 64 B per row
    const bool wide = RM && !ws && h->opt_rm_wide > 0;
    const bool tmem = wide || (RM && !ws && (h->opt_rm_tmem < 0 ? C::RM_TMEM : h->opt_rm_tmem > 0));
    int U = 0;
    auto kern = wide   ? pick_keystream_kernel<C, LAYOUT, RM, false, RM>(h, &U)
                : tmem ? pick_keystream_kernel<C, LAYOUT, RM>(h, &U)
                       : pick_keystream_kernel<C, LAYOUT>(h, &U);
    bsk::KsArgs a{};
    a.state = h->state;
    a.Gp = h->Gp;
    a.G = h->G;
    a.n = h->n;
    const uint64_t tail = h->n - (h->G - 1) * 32;
    a.tail_mask = tail >= 32 ? 0xFFFFFFFFu : ((1u << tail) - 1u);
    a.nclocks = bits;
    a.t0 = h->bits_done;
    a.g_base = h->first_instance / 32;
    a.out = out;
    a.row_bytes = bits / 8;
    a.units = h->units;
    a.scratch = h->sched + 1 + h->units;
    a.l2last = h->opt_rm_l2last;
    // staggered flush periods in the writer-warp kernel: auto = rows that are
    // not 16 B aligned (their pieces need 8 B stores whatever the phase)
    a.rm_phase = h->opt_rm_phase < 0 ? int(a.row_bytes % 16 != 0) : h->opt_rm_phase;

    int block = KS_BLOCK, compute_warps = KS_BLOCK / 32;
    size_t smem = RM ? size_t(KS_BLOCK / 32) * bsk::rm_warp_words(U, 8, true) * 4 : 0;
    if (tmem) smem = U == 32 ? 0 : size_t(KS_BLOCK / 32) * bsk::ZS_WORDS * 4;
    // TMA tensor stores for the whole-sector flushes of all-real warps: needs
    // 16 B aligned row strides (TMA global strides) and at least one such warp
    if (tmem && !wide && h->opt_rm_tma && (a.row_bytes % 16) == 0 && h->n / 32 >= 32 && a.row_bytes < (1ull << 32)) {
        if (int rc = encode_rowmajor_tmap(&a.tmap, out, a.row_bytes, h->n / 32)) return rc;
        a.use_tma = 1;
        a.tma_groups = h->n / 32;
        smem += size_t(KS_BLOCK / 32) * bsk::TMA_BUF_WORDS * 4;
    }
    if (ws) {
        kern = &bsk::keystream_rm_ws_kernel<C, C::U_DEFAULT>;
        if (h->opt_unroll == C::U_ALT0) kern = &bsk::keystream_rm_ws_kernel<C, C::U_ALT0>;
        if (h->opt_unroll == C::U_ALT1) kern = &bsk::keystream_rm_ws_kernel<C, C::U_ALT1>;
        block = bsk::ws::BLOCK;
        compute_warps = bsk::ws::NCOMP;
        smem = bsk::ws::SMEM_BYTES;
        // built for the output-bound ciphers only (C::RM_WS >= 2: the LFSR)
        if constexpr (C::RM_WS >= 2) {
            if (ws2) {
                kern = &bsk::keystream_rm_ws2_kernel<C, C::U_DEFAULT>;
                if (h->opt_unroll == C::U_ALT0) kern = &bsk::keystream_rm_ws2_kernel<C, C::U_ALT0>;
                if (h->opt_unroll == C::U_ALT1) kern = &bsk::keystream_rm_ws2_kernel<C, C::U_ALT1>;
                block = bsk::ws2::BLOCK;
                compute_warps = bsk::ws2::NSTREAM;
                smem = bsk::ws2::SMEM_BYTES;
            }
        } else if (ws2) {
            return fail(BSRNG_EINVAL, "rm_ws = 2 is built for the LFSR only");
        }
    }
    if (int rc = set_smem(reinterpret_cast<const void*>(kern), smem)) return rc;
    unsigned grid;
    int dbg_occ = 0, dbg_occ_max = 0;
    if (!persistent) {
        a.persistent = 0;
        a.nseg = 1;
        a.seg_clocks = bits;
        grid = unsigned((h->Gp + KS_BLOCK - 1) / KS_BLOCK);
    } else {
        int occ = h->opt_ctas_per_sm, occ_max = 1;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_max, kern, block, smem) != cudaSuccess ||
            occ_max < 1)
            occ_max = 1;
        // The occupancy API reports 1 CTA/SM for kernels that allocate tensor
        // memory; registers (255 x 128 threads -> 2 CTAs) and TMEM (2 x 256 of
        // 512 columns) allow two, which the GPU then runs (ncu: 7.9 warps/SM).
        if (tmem) occ_max = wide ? 1 : 2;
        // Auto policy (opt_ctas_per_sm == 0).  Many more warp-units than warp
        // slots: two warps per SMSP, one item per unit (no time segments, so no
        // warp ever waits on another; a warp left alone at the end runs at
        // nearly full rate).  Otherwise: one warp per SMSP and time segments,
        // so the tail is one segment long (with two warps per SMSP the issue
        // arbiter starves one of them and segment hand-offs stall).
        bool whole_units = false;
        if (occ <= 0) {
            const uint64_t slots2 = uint64_t(h->num_sms) * 2 * compute_warps;
            whole_units = !ws && occ_max >= 2 && h->units >= 3 * slots2 && !(tmem && C::RM_SEGMENTED);
            occ = (whole_units || tmem) ? 2 : 1;
        }
        if (wide) occ = 1;
        // an explicit setting is honoured even above the occupancy API's
        // estimate (extra CTAs queue; the ticket order cannot deadlock)
        if (occ > occ_max && h->opt_ctas_per_sm <= 0) occ = occ_max;
        dbg_occ = occ;
        dbg_occ_max = occ_max;
        const uint64_t slots = uint64_t(h->num_sms) * occ * compute_warps;  // resident clock-loop warps
        uint64_t nseg = 1;
        if (h->opt_seg_clocks) {
            nseg = (bits + h->opt_seg_clocks - 1) / h->opt_seg_clocks;
        } else if (!whole_units && h->units > slots) {
            // >= ~32 items per resident warp so the tail is <~3% of the call,
            // but segments no shorter than 256 clocks (state carry stays <1%)
            // (TMEM-staged ROW_MAJOR at two warps per SMSP: ~8 items per warp)
            const uint64_t per_warp = (tmem && !wide) ? 8 : 32;
            nseg = std::max<uint64_t>(1, (per_warp * slots + h->units - 1) / h->units);
            nseg = std::min<uint64_t>(nseg, std::max<uint64_t>(1, bits / 256));
        }
        nseg = std::max<uint64_t>(nseg, (bits + MAX_SEG_CLOCKS - 1) / MAX_SEG_CLOCKS);
        // whole 256-clock blocks keep ROW_MAJOR sector flushes full (32 B/row;
        // 512 clocks = 64 B for the wide staging)
        const uint64_t q_full = ws2 ? 1024 : (wide || ws) ? 512 : 256;
        const uint64_t quantum = bits >= q_full ? q_full : 32;
        uint64_t seg = ((bits + nseg - 1) / nseg + quantum - 1) / quantum * quantum;
        nseg = (bits + seg - 1) / seg;
        a.persistent = 1;
        a.nseg = nseg;
        a.seg_clocks = seg;
        a.ticket = h->sched;
        a.flags = h->sched + 1;
        const uint64_t items = h->units * nseg;
        const uint64_t want_ctas = ws ? items : (items * 32 + KS_BLOCK - 1) / KS_BLOCK;
        grid = unsigned(std::min<uint64_t>(want_ctas, uint64_t(h->num_sms) * occ));
        cudaError_t e = cudaMemsetAsync(h->sched, 0, (1 + h->units) * sizeof(uint32_t), st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset(sched): %s", cudaGetErrorString(e));
    }
    // one CTA per SM and no time segments (no CTA ever waits on another, so a
    // second CTA queued behind a 512-column allocation cannot deadlock): the
    // lone clock-loop warps get double-buffered TMEM staging (KsArgs::tmem_dbl)
    if constexpr (RM) {
        if (tmem && !wide && !a.use_tma && h->opt_rm_dbl && a.nseg == 1 && grid <= unsigned(h->num_sms)) {
            a.tmem_dbl = 1;
            kern = pick_keystream_kernel<C, LAYOUT, true, true>(h, &U);
            if (int rc = set_smem(reinterpret_cast<const void*>(kern), smem)) return rc;
        }
    }
    if (LAYOUT == bsk::L_CHECKSUM) {
        cudaError_t e = cudaMemsetAsync(out, 0, sizeof(uint64_t), st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset(out): %s", cudaGetErrorString(e));
    }
    static const bool debug = getenv("BSRNG_DEBUG") != nullptr;
    unsigned long long* dbg = nullptr;
    if (debug && a.persistent) {
        cudaMalloc(&dbg, 4 * sizeof(unsigned long long));
        cudaMemsetAsync(dbg, 0, 4 * sizeof(unsigned long long), st);
        a.dbg = dbg;
    }
    kern<<<grid, block, smem, st>>>(a);
    int rc = check_launch("keystream");
    if (dbg) {
        unsigned long long c[4];
        cudaMemcpyAsync(c, dbg, sizeof c, cudaMemcpyDeviceToHost, st);
        cudaStreamSynchronize(st);
        fprintf(stderr,
                "[bsrng] occ=%d/%d smem=%zu grid=%u units=%llu nseg=%llu seg=%llu tmem=%d dbl=%d tma=%d: "
                "waits=%llu slept=%llu spins=%llu\n",
                dbg_occ, dbg_occ_max, smem, grid, (unsigned long long)a.units, (unsigned long long)a.nseg,
                (unsigned long long)a.seg_clocks, int(tmem), a.tmem_dbl, a.use_tma, c[0], c[1], c[2]);
        cudaFree(dbg);
    }
    return rc;
}

template <class C>
int generate_stream_cipher(bsrng_t* h, void* out, uint64_t bits, bsrng_layout layout, cudaStream_t st)
{
    switch (layout) {
    case BSRNG_ROW_MAJOR: return launch_keystream<C, bsk::L_ROW_MAJOR>(h, out, bits, st);
    case BSRNG_SLICED: return launch_keystream<C, bsk::L_SLICED>(h, out, bits, st);
    case BSRNG_CHECKSUM: return launch_keystream<C, bsk::L_CHECKSUM>(h, out, bits, st);
    }
    return fail(BSRNG_EINVAL, "unknown layout %d", int(layout));
}

}  // namespace bsrng_impl
