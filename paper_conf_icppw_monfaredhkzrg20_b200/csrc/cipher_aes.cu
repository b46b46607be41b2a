// cipher_aes.cu -- AES-128-CTR (sec. 2.3.2; FIPS-197 [35];
// SURVEY NEXT-2): counter slicing, key expansion and keystream launches of
// libbsrng.so.  Kernels: aes.cuh.
#include <algorithm>
#include <mutex>

#include "aes.cuh"
#include "bitslice.cuh"
#include "internal.h"

namespace bsrng_impl {

namespace {
std::mutex g_slot_mu;
bool g_slot_used[bsk::aes::RK_SLOTS] = {};
}  // namespace

int aes_acquire_slot()
{
    std::lock_guard<std::mutex> lk(g_slot_mu);
    for (int i = 0; i < bsk::aes::RK_SLOTS; ++i)
        if (!g_slot_used[i]) {
            g_slot_used[i] = true;
            return i;
        }
    return -1;
}

void aes_release_slot(int slot)
{
    std::lock_guard<std::mutex> lk(g_slot_mu);
    if (slot >= 0 && slot < bsk::aes::RK_SLOTS) g_slot_used[slot] = false;
}

namespace {

int init_aes(bsrng_t* h, cudaStream_t st, const uint8_t* raw_k, const uint8_t* raw_iv, uint64_t g_split)
{
    // initial counter blocks sliced straight into the state rows (FIPS-197
    // bit order: bit 0 = MSB of byte 0); round keys from the one key.
    if (h->opt_init_fused) {
        if (int rc = set_smem(reinterpret_cast<const void*>(bsk::slice_state_kernel<16, 128, true>),
                              bsk::ss_smem_bytes(16)))
            return rc;
        bsk::slice_state_kernel<16, 128, true><<<unsigned((h->Gp + 127) / 128), 128, bsk::ss_smem_bytes(16), st>>>(
            raw_iv, h->tail + h->tail_iv_off, g_split, h->state, h->Gp);
    } else if (g_split >= h->Gp) {
        const unsigned sblocks = unsigned((h->Gp + bsk::SLICE_GROUPS - 1) / bsk::SLICE_GROUPS);
        bsk::slice_bits_kernel<16, 128, true><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_iv, h->n, h->state, h->Gp);
    } else {
        return fail(BSRNG_EINVAL, "unfused init needs staged inputs");
    }
    if (int rc = check_launch("slice(ctr)")) return rc;
    bsk::aes::aes_key_expand_kernel<<<1, 32, 0, st>>>(raw_k, h->rk_dev);
    if (int rc = check_launch("aes_key_expand")) return rc;
    // stream-ordered device-to-device copy into the handle's constant slot:
    // no host synchronisation on a rekey
    cudaError_t e = cudaMemcpyToSymbolAsync(bsk::aes::c_rk, h->rk_dev, sizeof(bsk::aes::RoundKeys),
                                            size_t(h->aes_slot) * sizeof(bsk::aes::RoundKeys),
                                            cudaMemcpyDeviceToDevice, st);
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "round keys: %s", cudaGetErrorString(e));
    return BSRNG_OK;
}

// Persistent grid, items = (time segment, warp-unit), independent (aes.cuh).
template <int LAYOUT>
int launch_aes(bsrng_t* h, void* out, uint64_t bits, cudaStream_t st, uint64_t row_stride = 0, uint64_t t0_add = 0)
{
    auto kern = &bsk::aes_ctr_kernel<LAYOUT>;
    bsk::KsArgs a{};
    a.state = h->state;
    a.Gp = h->Gp;
    a.G = h->G;
    a.n = h->n;
    const uint64_t tail = h->n - (h->G - 1) * 32;
    a.tail_mask = tail >= 32 ? 0xFFFFFFFFu : ((1u << tail) - 1u);
    a.nclocks = bits;
    a.t0 = h->bits_done + t0_add;
    a.g_base = h->first_instance / 32;
    a.out = out;
    a.row_bytes = row_stride ? row_stride : bits / 8;
    a.units = h->units;
    a.scratch = h->sched + 1 + h->units;
    a.persistent = 1;
    a.ticket = h->sched;
    a.flags = h->sched + 1;
    const size_t smem = size_t(128) * 128 * 4 + (LAYOUT == bsk::L_ROW_MAJOR ? size_t(4) * bsk::OS_WORDS * 4 : 0);
    if (int rc = set_smem(reinterpret_cast<const void*>(kern), smem)) return rc;
    // Two warps per SMSP (two CTAs per SM) when shared memory allows: the
    // second warp hides the round-key constant loads (short-scoreboard stalls)
    // and AES work items never wait on each other, so the issue arbiter's
    // favouritism cannot stall the queue.  ROW_MAJOR's sector buffers limit
    // it to one CTA per SM.
    int occ = h->opt_ctas_per_sm > 0 ? h->opt_ctas_per_sm : 2;
    int occ_max = 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_max, kern, 128, smem) != cudaSuccess || occ_max < 1)
        occ_max = 1;
    occ = std::min(occ, occ_max);
    const uint64_t slots = uint64_t(h->num_sms) * occ * 4;
    // Items (segment, warp-unit) are independent, so the split only trades
    // the queue's tail against per-item overhead (state load, counter setup,
    // checksum fold).  With at least two warp-units per slot: ~100 items per
    // slot but no item shorter than 8 blocks (C2 4.29 vs 4.24 Tb/s at 32
    // items per slot; 1024-bit rekey calls 3.81 vs 3.73 as whole units);
    // fewer units than that (the paper shape) need the finer split for
    // parallelism (C4: 2-block items 3.69, 8-block 3.64 Tb/s).
    const bool many = h->units >= 2 * slots;
    const uint64_t quantum = bits >= 256 ? 256 : 128;
    const uint64_t min_seg = many && bits >= 1024 && !h->opt_seg_clocks ? 1024 : quantum;
    uint64_t nseg = h->opt_seg_clocks ? (bits + h->opt_seg_clocks - 1) / h->opt_seg_clocks
                                      : ((many ? 100 : 32) * slots + h->units - 1) / h->units;
    nseg = std::max<uint64_t>(1, std::min<uint64_t>(nseg, bits / min_seg));
    nseg = std::max<uint64_t>(nseg, (bits + MAX_SEG_CLOCKS - 1) / MAX_SEG_CLOCKS);
    const uint64_t seg = ((bits + nseg - 1) / nseg + quantum - 1) / quantum * quantum;
    a.nseg = (bits + seg - 1) / seg;
    a.seg_clocks = seg;
    cudaError_t e = cudaMemsetAsync(h->sched, 0, (1 + h->units) * sizeof(uint32_t), st);
    if (e == cudaSuccess && LAYOUT == bsk::L_CHECKSUM) {
        e = cudaMemsetAsync(out, 0, sizeof(uint64_t), st);
        if (e == cudaSuccess && a.nseg > 1)
            e = cudaMemsetAsync(h->state + uint64_t(bsk::aes::NSTATE) * h->Gp, 0, h->Gp * 4, st);
    }
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset: %s", cudaGetErrorString(e));
    const uint64_t items = h->units * a.nseg;
    const unsigned grid = unsigned(std::min<uint64_t>((items + 3) / 4, uint64_t(h->num_sms) * occ));
    kern<<<grid, 128, smem, st>>>(a, h->aes_slot);
    return check_launch("aes_ctr");
}

// AES ROW_MAJOR with >= 32 blocks per instance: block-lane kernel (aes.cuh).
int launch_aes_rowmajor_lanes(bsrng_t* h, void* out, uint64_t bits, cudaStream_t st, uint64_t row_stride,
                              uint32_t* ticket)
{
    auto kern = &bsk::aes_ctr_rowmajor_lanes_kernel;
    bsk::KsArgs a{};
    a.state = h->state;
    a.n = h->n;
    a.G = h->G;
    a.Gp = h->Gp;
    a.nclocks = bits;
    a.t0 = h->bits_done;
    a.out = out;
    a.row_bytes = row_stride;
    a.units = h->G;  // one warp = 32 instances = one group
    a.persistent = 1;
    a.ticket = ticket;
    a.flags = nullptr;  // items are independent
    int occ = h->opt_ctas_per_sm > 0 ? h->opt_ctas_per_sm : 2;
    int occ_max = 1;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ_max, kern, 128, 0) != cudaSuccess || occ_max < 1)
        occ_max = 1;
    occ = std::min(occ, occ_max);
    const uint64_t slots = uint64_t(h->num_sms) * occ * 4;
    const uint64_t quantum = 4096;  // one 32-block encryption per instance
    uint64_t nseg = h->opt_seg_clocks ? (bits + h->opt_seg_clocks - 1) / h->opt_seg_clocks
                                      : (32 * slots + a.units - 1) / a.units;
    nseg = std::max<uint64_t>(1, std::min<uint64_t>(nseg, (bits + quantum - 1) / quantum));
    const uint64_t seg = ((bits + nseg - 1) / nseg + quantum - 1) / quantum * quantum;
    a.nseg = (bits + seg - 1) / seg;
    a.seg_clocks = seg;
    cudaError_t e = cudaMemsetAsync(ticket, 0, sizeof(uint32_t), st);
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset: %s", cudaGetErrorString(e));
    const uint64_t items = a.units * a.nseg;
    const unsigned grid = unsigned(std::min<uint64_t>((items + 3) / 4, uint64_t(h->num_sms) * occ));
    kern<<<grid, 128, 0, st>>>(a, h->aes_slot);
    return check_launch("aes_ctr_rowmajor_lanes");
}

int generate_aes(bsrng_t* h, void* out, uint64_t bits, bsrng_layout layout, cudaStream_t st)
{
    if (layout == BSRNG_ROW_MAJOR && bits >= 4096 && h->opt_rm_ws) {
        // whole 32-block encryptions per instance in the block-lane kernel
        // (one instance per thread); a remainder of < 32 blocks would waste
        // most of an encryption's lanes there (the paper-shape 35-block call
        // ran at 0.44 of the roofline), so it goes to the instance-sliced
        // kernel, writing the rows' last bytes
        const uint64_t main_bits = bits / 4096 * 4096, rem = bits - main_bits;
        if (!rem) return launch_aes_rowmajor_lanes(h, out, main_bits, st, bits / 8, h->sched);
        // The remainder (few warp-units, one warp per SMSP, one CTA per SM:
        // 18% of a paper-shape call run alone) goes first, on the handle's side
        // stream, so the block-lane kernel's CTAs fill the SMSPs beside it.
        // The two write disjoint bytes of the rows and only read the state;
        // each has its own queue ticket.
        if (!h->side) {
            if (cudaStreamCreateWithFlags(&h->side, cudaStreamNonBlocking) != cudaSuccess ||
                cudaEventCreateWithFlags(&h->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&h->ev_join, cudaEventDisableTiming) != cudaSuccess)
                return fail(BSRNG_ECUDA, "side stream / events");
        }
        cudaError_t e = cudaEventRecord(h->ev_fork, st);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(h->side, h->ev_fork, 0);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "fork: %s", cudaGetErrorString(e));
        int rc = launch_aes<bsk::L_ROW_MAJOR>(h, static_cast<uint8_t*>(out) + main_bits / 8, rem, h->side, bits / 8,
                                              main_bits);
        const int rc2 = launch_aes_rowmajor_lanes(h, out, main_bits, st, bits / 8, h->sched + 1 + h->units + 32);
        e = cudaEventRecord(h->ev_join, h->side);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(st, h->ev_join, 0);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "join: %s", cudaGetErrorString(e));
        return rc != BSRNG_OK ? rc : rc2;
    }
    switch (layout) {
    case BSRNG_ROW_MAJOR: return launch_aes<bsk::L_ROW_MAJOR>(h, out, bits, st);
    case BSRNG_SLICED: return launch_aes<bsk::L_SLICED>(h, out, bits, st);
    case BSRNG_CHECKSUM: return launch_aes<bsk::L_CHECKSUM>(h, out, bits, st);
    }
    return fail(BSRNG_EINVAL, "unknown layout %d", int(layout));
}

}  // namespace

const CipherOps k_aes_ops = {bsk::aes::NSTATE, init_aes, generate_aes};

}  // namespace bsrng_impl
