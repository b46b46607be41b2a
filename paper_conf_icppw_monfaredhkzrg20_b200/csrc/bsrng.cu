// bsrng.cu -- host side of the C ABI declared in include/bsrng.h.
//
// Handle = device-resident sliced cipher state [NSTATE + 1][Gp] (HBM) plus
// scratch for key/IV slicing and the persistent scheduler.  Every entry point
// validates its arguments, switches to the handle's device, enqueues kernels on
// the caller's stream and reports errors through a thread-local string.
// There is no CPU fallback anywhere in this library.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "../../include/bsrng.h"
#include "bitslice.cuh"
#include "keystream.cuh"
#include "aes.cuh"
#include "grain.cuh"
#include "lfsr.cuh"
#include "mickey2.cuh"
#include "rowmajor_ws.cuh"

namespace {

thread_local std::string g_err;
std::atomic<uint64_t> g_launches{0};

int fail(int code, const char* fmt, ...)
{
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

constexpr int KS_BLOCK = 128;
// Clocks unrolled per loop iteration.  The MICKEY loop body is ~331
// instructions (5.3 KB of SASS) per clock; at U = 8 it is 42 KB, beyond the
// 32 KB L1.5 instruction cache (B300_MICROARCH "I-cache"), and ncu showed
// "no_instruction" as the top stall.  Selectable per handle ("unroll").
constexpr int KS_U_DEFAULT = 0;  // 0 = the cipher's default (MICKEY 4, Grain 32)
// keystream bits per key/IV: MICKEY 2.0's limit is 2^40;
// Grain and AES-CTR are only bounded by the 64-bit bit counter here.
uint64_t max_bits(bsrng_cipher c) { return c == BSRNG_MICKEY2 ? (1ull << 40) : (1ull << 62); }

struct DeviceGuard {
    int prev = -1;
    bool ok = true;
    explicit DeviceGuard(int dev)
    {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) ok = cudaSetDevice(dev) == cudaSuccess;
    }
    ~DeviceGuard()
    {
        int cur;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

}  // namespace

struct bsrng {
    bsrng_cipher cipher;
    int dev = 0;
    int num_sms = 148;
    uint64_t n = 0, G = 0, Gp = 0, units = 0;
    uint64_t first_instance = 0;
    uint32_t iv_bits = 80;
    uint32_t key_bytes = 10, iv_bytes = 10;
    uint64_t key_rows = 0;       // n, or 1 for AES-CTR (one key for all instances)
    uint64_t bits_done = 0;
    uint32_t* state = nullptr;   // [NSTATE + 1][Gp]
    uint32_t* sliced = nullptr;  // key [KB][Gp] then iv [IVB][Gp]
    uint8_t* raw = nullptr;      // keys [n][key_bytes] then ivs [n][iv_bytes] at raw + iv_off
    uint64_t iv_off = 0;         // per-instance regions padded to Gp*32 rows (zeroed), 16 B aligned
    uint32_t* sched = nullptr;   // [1 + units]: ticket, flags; then [32] scratch
    uint8_t* bounce = nullptr;   // generate_host staging
    uint32_t* rk_dev = nullptr;  // AES: round-key masks written by the key-expansion kernel
    // device-input rekeys read whole 32-instance groups straight from the
    // caller's arrays; the partial last group and the padding groups (< 32)
    // come from this zeroed buffer: keys [32 groups * 32][key_bytes], then IVs
    uint8_t* tail = nullptr;
    uint64_t tail_iv_off = 0;
    bsk::aes::RoundKeys rk;      // AES: host copy, passed by value as a kernel parameter
    uint64_t bounce_bytes = 0;
    // options
    int opt_sched = 1;
    uint64_t opt_seg_clocks = 0;
    // Resident CTAs per SM; 0 = auto (launch_keystream / launch_aes).
    int opt_ctas_per_sm = 0;
    int opt_unroll = KS_U_DEFAULT;
    // ROW_MAJOR kernel choice: -1 = auto (MICKEY: warp-specialised compute/
    // writer kernel; Grain: in-register transpose in the clock kernel; AES:
    // block-lane kernel for calls of >= 32 blocks), 1 = specialised, 0 = plain
    int opt_rm_ws = -1;
    // ROW_MAJOR sector-staging slots per row (4 or 8); 0 = auto.
    int opt_rm_slots = 0;
    // ROW_MAJOR, U = 32: z block in registers (1) or staged in smem (0).
    int opt_rm_zreg = 1;
    // ROW_MAJOR plain kernel: stage row segments in TMEM (1) or smem (0).
    int opt_rm_tmem = -1;  // -1 = the cipher's default (C::RM_TMEM)
    // TMEM-staged ROW_MAJOR: whole-sector flushes as TMA tensor stores (1) or
    // as 8 B global stores from the 16x256b read-back (0)
    int opt_rm_tma = 1;
    // TMEM-staged ROW_MAJOR with one CTA per SM: double-buffered staging with
    // the previous sector period flushed 4 rows per block (1) or not (0)
    int opt_rm_dbl = 1;
    // init: slicing fused into the init kernel (MICKEY, Grain) / per-thread group
    // slicing into the state (AES, LFSR) (1), or the ballot slice kernels (0).
    int opt_init_fused = 1;
};

namespace {

int nstate_of(bsrng_cipher c)
{
    switch (c) {
    case BSRNG_MICKEY2: return bsk::Mickey2::NSTATE;
    case BSRNG_GRAIN_V1: return bsk::Grain::NSTATE;
    case BSRNG_AES128_CTR: return bsk::aes::NSTATE;
    case BSRNG_LFSR128: return bsk::Lfsr128::NSTATE;
    default: return 0;
    }
}

int check_launch(const char* what)
{
    g_launches.fetch_add(1, std::memory_order_relaxed);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "%s launch failed: %s", what, cudaGetErrorString(e));
    return BSRNG_OK;
}

// slice + initialisation clocks into h->state.  Groups g < g_split are read
// from raw_k / raw_iv (+ g * 32 * bytes), the rest from h->tail; the staged
// path passes h->raw and g_split = Gp.
int run_init(bsrng_t* h, cudaStream_t st, const uint8_t* raw_k, const uint8_t* raw_iv, uint64_t g_split)
{
    static bool ss_attr = false;  // > 48 KB of dynamic smem (coalesced staging)
    if (!ss_attr) {
        cudaError_t e = cudaFuncSetAttribute(bsk::slice_state_kernel<16, 128, true>,
                                             cudaFuncAttributeMaxDynamicSharedMemorySize, int(bsk::ss_smem_bytes(16)));
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "smem attribute: %s", cudaGetErrorString(e));
        ss_attr = true;
    }
    const uint64_t kbits = uint64_t(h->key_bytes) * 8, ivbits = uint64_t(h->iv_bytes) * 8;
    uint32_t* key_s = h->sliced;
    uint32_t* iv_s = h->sliced + kbits * h->Gp;
    const uint8_t* tail_k = h->tail;
    const uint8_t* tail_iv = h->tail + h->tail_iv_off;
    const bool staged = g_split >= h->Gp;
    const unsigned sblocks = unsigned((h->Gp + bsk::SLICE_GROUPS - 1) / bsk::SLICE_GROUPS);
    switch (h->cipher) {
    case BSRNG_MICKEY2: {
        if (h->opt_init_fused) {
            // one kernel: slicing in shared memory + the 260 mixing clocks
            const unsigned blocks = unsigned((h->Gp + bsk::M2I_BLOCK - 1) / bsk::M2I_BLOCK);
            static bool attr = false;
            if (!attr) {
                cudaError_t e = cudaFuncSetAttribute(bsk::m2_init_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                     int(bsk::M2I_SMEM_BYTES));
                if (e != cudaSuccess) return fail(BSRNG_ECUDA, "smem attribute: %s", cudaGetErrorString(e));
                attr = true;
            }
            bsk::m2_init_kernel<<<blocks, bsk::M2I_BLOCK, bsk::M2I_SMEM_BYTES, st>>>(
                raw_k, raw_iv, tail_k, tail_iv, g_split, int(h->iv_bits), h->state, h->Gp);
            return check_launch("m2_init");
        }
        if (!staged) return fail(BSRNG_EINVAL, "unfused init needs staged inputs");
        bsk::slice_bits_kernel<10, 80, true><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_k, h->n, key_s, h->Gp);
        if (int rc = check_launch("slice(key)")) return rc;
        bsk::slice_bits_kernel<10, 80, true><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_iv, h->n, iv_s, h->Gp);
        if (int rc = check_launch("slice(iv)")) return rc;
        const unsigned pblocks = unsigned((h->Gp + 127) / 128);
        bsk::m2_preclock_kernel<<<pblocks, 128, 0, st>>>(iv_s, key_s, int(h->iv_bits), h->state, h->Gp);
        if (int rc = check_launch("m2_preclock")) return rc;
        (void)ivbits;
        return BSRNG_OK;
    }
    case BSRNG_GRAIN_V1: {
        // spec [15]: key and IV bits are taken LSB-first from their bytes
        if (h->opt_init_fused) {
            const unsigned blocks = unsigned((h->Gp + 127) / 128);
            static bool gattr = false;
            if (!gattr) {
                cudaError_t e = cudaFuncSetAttribute(bsk::grain_init_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                     int(bsk::GI_SMEM_BYTES));
                if (e != cudaSuccess) return fail(BSRNG_ECUDA, "smem attribute: %s", cudaGetErrorString(e));
                gattr = true;
            }
            bsk::grain_init_kernel<<<unsigned((h->Gp + GI_BLOCK - 1) / GI_BLOCK), GI_BLOCK, bsk::GI_SMEM_BYTES, st>>>(
                raw_k, raw_iv, tail_k, tail_iv, g_split,
                                                                           h->state, h->Gp);
            return check_launch("grain_init");
        }
        if (!staged) return fail(BSRNG_EINVAL, "unfused init needs staged inputs");
        bsk::slice_bits_kernel<10, 80, false><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_k, h->n, key_s, h->Gp);
        if (int rc = check_launch("slice(key)")) return rc;
        bsk::slice_bits_kernel<8, 64, false><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_iv, h->n, iv_s, h->Gp);
        if (int rc = check_launch("slice(iv)")) return rc;
        const unsigned pblocks = unsigned((h->Gp + 127) / 128);
        bsk::grain_preclock_kernel<<<pblocks, 128, 0, st>>>(key_s, iv_s, h->state, h->Gp);
        return check_launch("grain_preclock");
    }
    case BSRNG_AES128_CTR: {
        // initial counter blocks sliced straight into the state rows (FIPS-197
        // bit order: bit 0 = MSB of byte 0); round keys from the one key.
        if (h->opt_init_fused)
            bsk::slice_state_kernel<16, 128, true><<<unsigned((h->Gp + 127) / 128), 128, bsk::ss_smem_bytes(16), st>>>(
                raw_iv, tail_iv, g_split, h->state, h->Gp);
        else if (staged)
            bsk::slice_bits_kernel<16, 128, true><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_iv, h->n, h->state, h->Gp);
        else
            return fail(BSRNG_EINVAL, "unfused init needs staged inputs");
        if (int rc = check_launch("slice(ctr)")) return rc;
        bsk::aes::aes_key_expand_kernel<<<1, 32, 0, st>>>(raw_k, h->rk_dev);
        if (int rc = check_launch("aes_key_expand")) return rc;
        // the masks become kernel parameters (constant-bank LOP3 operands): one
        // small synchronous D2H copy per rekey
        cudaError_t e = cudaMemcpyAsync(&h->rk, h->rk_dev, sizeof(h->rk), cudaMemcpyDeviceToHost, st);
        if (e == cudaSuccess) e = cudaStreamSynchronize(st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "round keys: %s", cudaGetErrorString(e));
        (void)key_s;
        (void)iv_s;
        return BSRNG_OK;
    }
    case BSRNG_LFSR128: {
        // the state IS the key: 128 bits, MSB-first, sliced straight into rows 0..127
        if (h->opt_init_fused)
            bsk::slice_state_kernel<16, 128, true><<<unsigned((h->Gp + 127) / 128), 128, bsk::ss_smem_bytes(16), st>>>(
                raw_k, tail_k, g_split, h->state, h->Gp);
        else if (staged)
            bsk::slice_bits_kernel<16, 128, true><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_k, h->n, h->state, h->Gp);
        else
            return fail(BSRNG_EINVAL, "unfused init needs staged inputs");
        if (int rc = check_launch("slice(key)")) return rc;
        cudaError_t e = cudaMemsetAsync(h->state + uint64_t(bsk::Lfsr128::NSTATE) * h->Gp, 0, h->Gp * 4, st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset: %s", cudaGetErrorString(e));
        (void)key_s;
        (void)iv_s;
        return BSRNG_OK;
    }
    default: return fail(BSRNG_EUNSUPPORTED, "cipher %d not built", int(h->cipher));
    }
}

int copy_inputs(bsrng_t* h, const uint8_t* keys, const uint8_t* ivs, uint32_t flags, cudaStream_t st)
{
    const size_t kb = size_t(h->key_rows) * h->key_bytes, vb = size_t(h->n) * h->iv_bytes;
    const cudaMemcpyKind kind = (flags & BSRNG_INPUT_DEVICE) ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    cudaError_t e = cudaMemcpyAsync(h->raw, keys, kb, kind, st);
    if (e == cudaSuccess && vb) e = cudaMemcpyAsync(h->raw + h->iv_off, ivs, vb, kind, st);
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "key/iv copy failed: %s", cudaGetErrorString(e));
    return BSRNG_OK;
}

// Tensor map for TMA ROW_MAJOR flushes (keystream.cuh rowmajor_store_tmem_tma):
// element (byte c, group g, q) of the 3-D view = out[(32 g + q) * row_bytes + c],
// dims {row_bytes, groups, 32}, box {32 B, 8 groups, 32}.  The driver's
// cuTensorMapEncodeTiled is reached through the runtime's entry-point query
// (no libcuda link dependency).
using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int encode_rowmajor_tmap(CUtensorMap* map, void* out, uint64_t row_bytes, uint64_t groups)
{
    static EncodeTiledFn encode = nullptr;
    if (!encode) {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess || !fn)
            return fail(BSRNG_ECUDA, "cuTensorMapEncodeTiled unavailable");
        encode = reinterpret_cast<EncodeTiledFn>(fn);
    }
    const cuuint64_t dims[3] = {row_bytes, groups, 32};
    const cuuint64_t strides[2] = {32 * row_bytes, row_bytes};
    const cuuint32_t box[3] = {32, 8, 32}, estr[3] = {1, 1, 1};
    const CUresult r = encode(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, out, dims, strides, box, estr,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                              CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return fail(BSRNG_ECUDA, "cuTensorMapEncodeTiled failed (%d)", int(r));
    return BSRNG_OK;
}

// Kernel instance for the handle's unroll option and ROW_MAJOR staging slots.
template <class C, int LAYOUT, int SLOTS, bool ZREG = true, bool TMEM = false, bool DBL = false>
auto pick_keystream_kernel(const bsrng_t* h, int* U)
{
    auto kern = &bsk::keystream_kernel<C, LAYOUT, C::U_DEFAULT, KS_BLOCK, SLOTS, ZREG, TMEM, DBL>;
    *U = C::U_DEFAULT;
    if (h->opt_unroll == C::U_ALT0)
        kern = &bsk::keystream_kernel<C, LAYOUT, C::U_ALT0, KS_BLOCK, SLOTS, true, TMEM, DBL>, *U = C::U_ALT0;
    if (h->opt_unroll == C::U_ALT1)
        kern = &bsk::keystream_kernel<C, LAYOUT, C::U_ALT1, KS_BLOCK, SLOTS, true, TMEM, DBL>, *U = C::U_ALT1;
    return kern;
}

template <class C, int LAYOUT>
int launch_keystream(bsrng_t* h, void* out, uint64_t bits, cudaStream_t st)
{
    // ROW_MAJOR row-segment staging: 8 slots (whole 32 B sectors, default) or
    // 4 (16 B, half the shared memory; ncu: L2 then fetches and re-evicts the
    // half-written sectors, ~3x the algorithmic DRAM traffic).
    int slots = h->opt_rm_slots ? h->opt_rm_slots : 8;
    if (LAYOUT != bsk::L_ROW_MAJOR) slots = 8;
    // U = 32 loops keep the 32-clock z block in registers (zreg) or stage it
    // in shared memory one word per clock (fewer live registers).
    const bool zreg = LAYOUT != bsk::L_ROW_MAJOR || h->opt_rm_zreg != 0;
    // ROW_MAJOR kernel: warp-specialised compute/writer kernel (rowmajor_ws.cuh,
    // 8 warps per CTA of which 4 run the clock loop; always persistent), or
    // the plain clock kernel with the row segments staged in tensor memory
    // (TMEM) or shared memory.  Defaults per cipher (RM_TMEM traits).
    const bool ws_pref = h->opt_rm_ws < 0 ? (C::U_DEFAULT != 32 && !C::RM_TMEM) : (h->opt_rm_ws != 0);
    const bool ws = LAYOUT == bsk::L_ROW_MAJOR && ws_pref && h->opt_sched != 0;
    const bool tmem = LAYOUT == bsk::L_ROW_MAJOR && !ws && (h->opt_rm_tmem < 0 ? C::RM_TMEM : h->opt_rm_tmem > 0);
    int U = 0;
    auto kern = pick_keystream_kernel<C, LAYOUT, 8>(h, &U);
    if (tmem) {
        kern = zreg ? pick_keystream_kernel<C, LAYOUT, 8, true, true>(h, &U)
                    : pick_keystream_kernel<C, LAYOUT, 8, false, true>(h, &U);
    } else if (LAYOUT == bsk::L_ROW_MAJOR) {
        if (slots == 4 && zreg) kern = pick_keystream_kernel<C, LAYOUT, 4>(h, &U);
        if (slots == 4 && !zreg) kern = pick_keystream_kernel<C, LAYOUT, 4, false>(h, &U);
        if (slots == 8 && !zreg) kern = pick_keystream_kernel<C, LAYOUT, 8, false>(h, &U);
    }
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

    int block = KS_BLOCK, compute_warps = KS_BLOCK / 32;
    size_t smem = LAYOUT == bsk::L_ROW_MAJOR ? size_t(KS_BLOCK / 32) * bsk::rm_warp_words(U, slots, zreg) * 4 : 0;
    if (tmem) smem = (U == 32 && zreg) ? 0 : size_t(KS_BLOCK / 32) * bsk::ZS_WORDS * 4;
    // TMA tensor stores for the whole-sector flushes of all-real warps: needs
    // 16 B aligned row strides (TMA global strides) and at least one such warp
    if (tmem && h->opt_rm_tma && (a.row_bytes % 16) == 0 && h->n / 32 >= 32 && a.row_bytes < (1ull << 32)) {
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
    }
    if (smem > 48 * 1024) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "smem attribute: %s", cudaGetErrorString(e));
    }
    unsigned grid;
    int dbg_occ = 0, dbg_occ_max = 0;
    if (h->opt_sched == 0) {
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
        if (tmem) occ_max = 2;
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
            const uint64_t per_warp = tmem ? 8 : 32;
            nseg = std::max<uint64_t>(1, (per_warp * slots + h->units - 1) / h->units);
            nseg = std::min<uint64_t>(nseg, std::max<uint64_t>(1, bits / 256));
        }
        // whole 256-clock blocks keep ROW_MAJOR sector flushes full (32 B/row)
        const uint64_t quantum = bits >= 256 ? 256 : 32;
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
    if (LAYOUT == bsk::L_ROW_MAJOR && tmem && !a.use_tma && h->opt_rm_dbl && a.nseg == 1 &&
        grid <= unsigned(h->num_sms)) {
        a.tmem_dbl = 1;
        kern = zreg ? pick_keystream_kernel<C, LAYOUT, 8, true, true, true>(h, &U)
                    : pick_keystream_kernel<C, LAYOUT, 8, false, true, true>(h, &U);
        if (smem > 48 * 1024) {
            cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
            if (e != cudaSuccess) return fail(BSRNG_ECUDA, "smem attribute: %s", cudaGetErrorString(e));
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
        fprintf(stderr, "[bsrng] occ=%d/%d smem=%zu grid=%u units=%llu nseg=%llu seg=%llu: waits=%llu slept=%llu spins=%llu\n",
                dbg_occ, dbg_occ_max, smem, grid,
                (unsigned long long)a.units, (unsigned long long)a.nseg, (unsigned long long)a.seg_clocks, c[0], c[1],
                c[2]);
        cudaFree(dbg);
    }
    return rc;
}

// AES-CTR: persistent grid of one 4-warp CTA per SM; work items (time segment,
// warp-unit) are independent, so segments need no flags (aes.cuh).
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
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "smem attribute: %s", cudaGetErrorString(e));
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
    const uint64_t quantum = bits >= 256 ? 256 : 128;
    uint64_t nseg = h->opt_seg_clocks ? (bits + h->opt_seg_clocks - 1) / h->opt_seg_clocks
                                      : (32 * slots + h->units - 1) / h->units;
    nseg = std::max<uint64_t>(1, std::min<uint64_t>(nseg, bits / quantum));
    const uint64_t seg = ((bits + nseg - 1) / nseg + quantum - 1) / quantum * quantum;
    a.nseg = (bits + seg - 1) / seg;
    a.seg_clocks = seg;
    e = cudaMemsetAsync(h->sched, 0, (1 + h->units) * sizeof(uint32_t), st);
    if (e == cudaSuccess && LAYOUT == bsk::L_CHECKSUM) {
        e = cudaMemsetAsync(out, 0, sizeof(uint64_t), st);
        if (e == cudaSuccess && a.nseg > 1)
            e = cudaMemsetAsync(h->state + uint64_t(bsk::aes::NSTATE) * h->Gp, 0, h->Gp * 4, st);
    }
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset: %s", cudaGetErrorString(e));
    const uint64_t items = h->units * a.nseg;
    const unsigned grid = unsigned(std::min<uint64_t>((items + 3) / 4, uint64_t(h->num_sms) * occ));
    kern<<<grid, 128, smem, st>>>(a, h->rk);
    return check_launch("aes_ctr");
}

// AES ROW_MAJOR with >= 32 blocks per instance: block-lane kernel (aes.cuh).
int launch_aes_rowmajor_lanes(bsrng_t* h, void* out, uint64_t bits, cudaStream_t st, uint64_t row_stride = 0)
{
    auto kern = &bsk::aes_ctr_rowmajor_lanes_kernel;
    bsk::KsArgs a{};
    a.n = h->n;
    a.G = h->G;
    a.Gp = h->Gp;
    a.nclocks = bits;
    a.t0 = h->bits_done;
    a.out = out;
    a.row_bytes = row_stride ? row_stride : bits / 8;
    a.units = h->G;  // one warp = 32 instances
    a.aux = h->raw + h->iv_off;
    a.persistent = 1;
    a.ticket = h->sched;
    a.flags = h->sched + 1;
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
    cudaError_t e = cudaMemsetAsync(h->sched, 0, sizeof(uint32_t), st);
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset: %s", cudaGetErrorString(e));
    const uint64_t items = a.units * a.nseg;
    const unsigned grid = unsigned(std::min<uint64_t>((items + 3) / 4, uint64_t(h->num_sms) * occ));
    kern<<<grid, 128, 0, st>>>(a, h->rk);
    return check_launch("aes_ctr_rowmajor_lanes");
}

template <class C>
int dispatch_layout(bsrng_t* h, void* out, uint64_t bits, bsrng_layout layout, cudaStream_t st)
{
    switch (layout) {
    case BSRNG_ROW_MAJOR: return launch_keystream<C, bsk::L_ROW_MAJOR>(h, out, bits, st);
    case BSRNG_SLICED: return launch_keystream<C, bsk::L_SLICED>(h, out, bits, st);
    case BSRNG_CHECKSUM: return launch_keystream<C, bsk::L_CHECKSUM>(h, out, bits, st);
    }
    return fail(BSRNG_EINVAL, "unknown layout %d", int(layout));
}

int validate_generate(const bsrng_t* h, const void* out, uint64_t bits, bsrng_layout layout, bool host)
{
    if (!h) return fail(BSRNG_EINVAL, "NULL handle");
    if (!out) return fail(BSRNG_EINVAL, "NULL out");
    if (layout != BSRNG_ROW_MAJOR && layout != BSRNG_SLICED && layout != BSRNG_CHECKSUM)
        return fail(BSRNG_EINVAL, "unknown layout %d", int(layout));
    const uint64_t q = h->cipher == BSRNG_AES128_CTR ? 128 : 32;
    if (bits % q != 0)
        return fail(BSRNG_EINVAL, "bits_per_instance=%llu is not a multiple of %llu", (unsigned long long)bits,
                    (unsigned long long)q);
    const uintptr_t align = layout == BSRNG_CHECKSUM ? 8 : 16;
    if (!host && (reinterpret_cast<uintptr_t>(out) % align) != 0)
        return fail(BSRNG_EINVAL, "out is not %u-byte aligned", unsigned(align));
    const uint64_t lim = max_bits(h->cipher);
    if (bits > lim || h->bits_done + bits > lim)
        return fail(BSRNG_ERANGE, "cumulative keystream would exceed %s bits per key/IV",
                    h->cipher == BSRNG_MICKEY2 ? "2^40" : "2^62");
    return BSRNG_OK;
}

}  // namespace

extern "C" {

const char* bsrng_last_error(void) { return g_err.c_str(); }

uint64_t bsrng_launch_count(void) { return g_launches.load(); }

bsrng_t* bsrng_create_ex(bsrng_cipher cipher, const uint8_t* keys, const uint8_t* ivs, uint32_t iv_bits,
                         uint64_t n, uint64_t first_instance_id, uint32_t flags, void* stream)
{
    g_err.clear();
    if (nstate_of(cipher) == 0) {
        fail(BSRNG_EINVAL, "cipher %d not supported", int(cipher));
        return nullptr;
    }
    if (cipher == BSRNG_AES128_CTR && iv_bits != 128) {
        fail(BSRNG_EINVAL, "AES-128-CTR iv_bits=%u must be 128 (one 16-byte counter block per instance)", iv_bits);
        return nullptr;
    }
    if (!keys || (!ivs && iv_bits > 0)) { fail(BSRNG_EINVAL, "NULL keys/ivs"); return nullptr; }
    if (n == 0) { fail(BSRNG_EINVAL, "n_instances == 0"); return nullptr; }
    if (first_instance_id % 32) { fail(BSRNG_EINVAL, "first_instance_id must be a multiple of 32"); return nullptr; }
    if (flags & ~uint32_t(BSRNG_INPUT_DEVICE)) { fail(BSRNG_EINVAL, "unknown flags 0x%x", flags); return nullptr; }
    if (cipher == BSRNG_LFSR128 && iv_bits != 0) {
        fail(BSRNG_EINVAL, "LFSR iv_bits=%u must be 0 (the state is the key)", iv_bits);
        return nullptr;
    }
    if (cipher == BSRNG_GRAIN_V1 && iv_bits != 64) {
        fail(BSRNG_EINVAL, "Grain v1 iv_bits=%u must be 64", iv_bits);
        return nullptr;
    }
    if (cipher == BSRNG_MICKEY2 && (iv_bits > 80 || iv_bits % 8)) {
        fail(BSRNG_EINVAL, "MICKEY iv_bits=%u must be a multiple of 8 in [0, 80]", iv_bits);
        return nullptr;
    }
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { fail(BSRNG_ECUDA, "no CUDA device"); return nullptr; }
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, dev) != cudaSuccess) { fail(BSRNG_ECUDA, "cudaGetDeviceProperties failed"); return nullptr; }
    if (prop.major != 10) {
        fail(BSRNG_ECUDA, "device %d is sm_%d%d; this library is built for sm_100a only", dev, prop.major, prop.minor);
        return nullptr;
    }
    bsrng_t* h = new bsrng_t();
    h->cipher = cipher;
    h->dev = dev;
    h->num_sms = prop.multiProcessorCount;
    h->n = n;
    h->G = (n + 31) / 32;
    h->units = (h->G + 31) / 32;
    h->Gp = h->units * 32;
    h->first_instance = first_instance_id;
    h->iv_bits = iv_bits;
    const bool aes = cipher == BSRNG_AES128_CTR, lfsr = cipher == BSRNG_LFSR128;
    h->key_bytes = (aes || lfsr) ? 16 : 10;
    h->iv_bytes = cipher == BSRNG_GRAIN_V1 ? 8 : aes ? 16 : lfsr ? 0 : 10;
    h->key_rows = aes ? 1 : h->n;
    // the fused init kernels read whole 32-instance group blocks with 16 B
    // loads: the per-instance regions are padded to Gp*32 rows and zeroed
    h->iv_off = aes ? 16 : h->Gp * 32 * h->key_bytes;  // AES: one 16 B key
    const uint64_t raw_bytes = h->iv_off + h->Gp * 32 * h->iv_bytes;
    const int ns = nstate_of(cipher);
    const uint64_t sl_words = (aes || lfsr) ? 1 : uint64_t(h->key_bytes + h->iv_bytes) * 8 * h->Gp;
    if (cudaMalloc(&h->state, uint64_t(ns + 1) * h->Gp * 4) != cudaSuccess ||
        cudaMalloc(&h->sliced, sl_words * 4) != cudaSuccess ||
        cudaMalloc(&h->raw, raw_bytes) != cudaSuccess ||
        cudaMalloc(&h->sched, (1 + h->units + 32) * 4) != cudaSuccess ||
        (aes && cudaMalloc(&h->rk_dev, sizeof(bsk::aes::RoundKeys)) != cudaSuccess) ||
        cudaMalloc(&h->tail, 32 * 32 * uint64_t(h->key_bytes + h->iv_bytes)) != cudaSuccess) {
        cudaGetLastError();
        bsrng_destroy(h);
        fail(BSRNG_ENOMEM, "cudaMalloc failed for %llu instances", (unsigned long long)n);
        return nullptr;
    }
    h->tail_iv_off = 32 * 32 * uint64_t(h->key_bytes);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (cudaMemsetAsync(h->raw, 0, raw_bytes, st) != cudaSuccess ||
        cudaMemsetAsync(h->tail, 0, 32 * 32 * uint64_t(h->key_bytes + h->iv_bytes), st) != cudaSuccess) {
        bsrng_destroy(h);
        fail(BSRNG_ECUDA, "memset(raw) failed");
        return nullptr;
    }
    if (bsrng_rekey(h, keys, ivs, flags, stream) != BSRNG_OK) {
        std::string msg = g_err;
        bsrng_destroy(h);
        g_err = msg;
        return nullptr;
    }
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) {
        bsrng_destroy(h);
        fail(BSRNG_ECUDA, "init failed: %s", cudaGetErrorString(e));
        return nullptr;
    }
    return h;
}

bsrng_t* bsrng_create(bsrng_cipher cipher, const uint8_t* keys, const uint8_t* ivs, uint64_t n)
{
    const uint32_t ivb = cipher == BSRNG_GRAIN_V1 ? 64 : cipher == BSRNG_AES128_CTR ? 128 : cipher == BSRNG_LFSR128 ? 0 : 80;
    return bsrng_create_ex(cipher, keys, ivs, ivb, n, 0, BSRNG_INPUT_HOST, nullptr);
}

int bsrng_rekey(bsrng_t* h, const uint8_t* keys, const uint8_t* ivs, uint32_t flags, void* stream)
{
    if (!h) return fail(BSRNG_EINVAL, "NULL handle");
    if (!keys) return fail(BSRNG_EINVAL, "NULL keys");
    if (!ivs && h->iv_bits > 0) return fail(BSRNG_EINVAL, "NULL ivs");
    DeviceGuard dg(h->dev);
    if (!dg.ok) return fail(BSRNG_ECUDA, "cudaSetDevice(%d) failed", h->dev);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    // Device inputs, 16 B aligned, fused init: the init kernels read whole
    // groups straight from the caller's arrays (no staging copy, ~25 us per
    // 2^22 keys); only the partial last group goes through h->tail.
    const bool aes = h->cipher == BSRNG_AES128_CTR;
    const bool direct = (flags & BSRNG_INPUT_DEVICE) && h->opt_init_fused && h->tail && ivs &&
                        ((reinterpret_cast<uintptr_t>(keys) | reinterpret_cast<uintptr_t>(ivs)) & 15) == 0 &&
                        !(h->cipher == BSRNG_MICKEY2 && h->iv_bytes != 10);
    if (direct) {
        const uint64_t g_split = h->n / 32, rest = h->n - g_split * 32;
        cudaError_t e = cudaSuccess;
        if (rest) {
            if (!aes && h->key_bytes)
                e = cudaMemcpyAsync(h->tail, keys + g_split * 32 * h->key_bytes, rest * h->key_bytes,
                                    cudaMemcpyDeviceToDevice, st);
            if (e == cudaSuccess && h->iv_bytes)
                e = cudaMemcpyAsync(h->tail + h->tail_iv_off, ivs + g_split * 32 * h->iv_bytes, rest * h->iv_bytes,
                                    cudaMemcpyDeviceToDevice, st);
            if (e != cudaSuccess) return fail(BSRNG_ECUDA, "tail copy: %s", cudaGetErrorString(e));
        }
        if (int rc = run_init(h, st, keys, ivs, g_split)) return rc;
        h->bits_done = 0;
        return BSRNG_OK;
    }
    if (!ivs) {  // iv_bits == 0: IV bytes are never read; keep them defined
        cudaError_t e = cudaMemsetAsync(h->raw + h->iv_off, 0, h->n * h->iv_bytes, st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset: %s", cudaGetErrorString(e));
        const cudaMemcpyKind kind = (flags & BSRNG_INPUT_DEVICE) ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
        e = cudaMemcpyAsync(h->raw, keys, h->key_rows * h->key_bytes, kind, st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "key copy: %s", cudaGetErrorString(e));
    } else if (int rc = copy_inputs(h, keys, ivs, flags, st)) {
        return rc;
    }
    if (int rc = run_init(h, st, h->raw, h->raw + h->iv_off, h->Gp)) return rc;
    h->bits_done = 0;
    return BSRNG_OK;
}

int bsrng_generate(bsrng_t* h, void* out, uint64_t bits, bsrng_layout layout, void* stream)
{
    if (int rc = validate_generate(h, out, bits, layout, false)) return rc;
    if (bits == 0) return BSRNG_OK;
    DeviceGuard dg(h->dev);
    if (!dg.ok) return fail(BSRNG_ECUDA, "cudaSetDevice(%d) failed", h->dev);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    int rc;
    switch (h->cipher) {
    case BSRNG_MICKEY2: rc = dispatch_layout<bsk::Mickey2>(h, out, bits, layout, st); break;
    case BSRNG_GRAIN_V1: rc = dispatch_layout<bsk::Grain>(h, out, bits, layout, st); break;
    case BSRNG_LFSR128: rc = dispatch_layout<bsk::Lfsr128>(h, out, bits, layout, st); break;
    case BSRNG_AES128_CTR:
        if (layout == BSRNG_ROW_MAJOR && bits >= 4096 && h->opt_rm_ws) {
            // whole 32-block encryptions per instance in the block-lane kernel
            // (one instance per thread); a remainder of < 32 blocks would waste
            // most of an encryption's lanes there (the paper-shape 35-block
            // call ran at 0.44 of the roofline), so it goes to the
            // instance-sliced kernel, writing the rows' last bytes
            const uint64_t main_bits = bits / 4096 * 4096, rem = bits - main_bits;
            rc = launch_aes_rowmajor_lanes(h, out, main_bits, st, bits / 8);
            if (rc == BSRNG_OK && rem)
                rc = launch_aes<bsk::L_ROW_MAJOR>(h, static_cast<uint8_t*>(out) + main_bits / 8, rem, st, bits / 8,
                                                  main_bits);
        } else {
            rc = layout == BSRNG_ROW_MAJOR ? launch_aes<bsk::L_ROW_MAJOR>(h, out, bits, st)
                 : layout == BSRNG_SLICED  ? launch_aes<bsk::L_SLICED>(h, out, bits, st)
                                           : launch_aes<bsk::L_CHECKSUM>(h, out, bits, st);
        }
        break;
    default: rc = fail(BSRNG_EUNSUPPORTED, "cipher not built");
    }
    if (rc == BSRNG_OK) h->bits_done += bits;
    return rc;
}

uint64_t bsrng_out_bytes(const bsrng_t* h, uint64_t bits, bsrng_layout layout)
{
    if (!h) return 0;
    switch (layout) {
    case BSRNG_ROW_MAJOR: return h->n * (bits / 8);
    case BSRNG_SLICED: return bits * h->G * 4;
    case BSRNG_CHECKSUM: return 8;
    }
    return 0;
}

int bsrng_generate_host(bsrng_t* h, void* host_out, uint64_t bits, bsrng_layout layout, void* stream)
{
    if (int rc = validate_generate(h, host_out, bits, layout, true)) return rc;
    if (bits == 0) return BSRNG_OK;
    DeviceGuard dg(h->dev);
    if (!dg.ok) return fail(BSRNG_ECUDA, "cudaSetDevice(%d) failed", h->dev);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    // chunk so the device staging buffer stays <= 1 GiB
    const uint64_t cap = 1ull << 30;
    uint64_t per_clock = layout == BSRNG_ROW_MAJOR ? (h->n + 7) / 8 : layout == BSRNG_SLICED ? h->G * 4 : 0;
    uint64_t chunk = bits;
    const uint64_t cq = h->cipher == BSRNG_AES128_CTR ? 256 : 32;
    if (per_clock) chunk = std::max<uint64_t>(cq, std::min<uint64_t>(bits, cap / per_clock / cq * cq));
    if (layout == BSRNG_CHECKSUM) chunk = bits;  // a checksum covers the whole call
    const uint64_t need = bsrng_out_bytes(h, chunk, layout);
    if (h->bounce_bytes < need) {
        if (h->bounce) cudaFree(h->bounce);
        h->bounce = nullptr;
        h->bounce_bytes = 0;
        if (cudaMalloc(&h->bounce, need) != cudaSuccess) {
            cudaGetLastError();
            return fail(BSRNG_ENOMEM, "cudaMalloc(%llu) for host staging", (unsigned long long)need);
        }
        h->bounce_bytes = need;
    }
    uint8_t* dst = static_cast<uint8_t*>(host_out);
    for (uint64_t done = 0; done < bits; done += chunk) {
        const uint64_t c = std::min(chunk, bits - done);
        if (int rc = bsrng_generate(h, h->bounce, c, layout, stream)) return rc;
        cudaError_t e;
        if (layout == BSRNG_ROW_MAJOR)
            e = cudaMemcpy2DAsync(dst + done / 8, bits / 8, h->bounce, c / 8, c / 8, h->n,
                                  cudaMemcpyDeviceToHost, st);
        else if (layout == BSRNG_SLICED)
            e = cudaMemcpyAsync(dst + done * h->G * 4, h->bounce, c * h->G * 4, cudaMemcpyDeviceToHost, st);
        else
            e = cudaMemcpyAsync(dst, h->bounce, 8, cudaMemcpyDeviceToHost, st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "D2H copy: %s", cudaGetErrorString(e));
    }
    cudaError_t e = cudaStreamSynchronize(st);
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "generate_host: %s", cudaGetErrorString(e));
    return BSRNG_OK;
}

uint64_t bsrng_num_instances(const bsrng_t* h) { return h ? h->n : 0; }
uint64_t bsrng_num_groups(const bsrng_t* h) { return h ? h->G : 0; }
uint64_t bsrng_bits_done(const bsrng_t* h) { return h ? h->bits_done : 0; }

int64_t bsrng_copy_state(const bsrng_t* h, uint32_t* host_out, uint64_t words)
{
    if (!h || !host_out) return fail(BSRNG_EINVAL, "NULL argument");
    const uint64_t ns = uint64_t(nstate_of(h->cipher));
    const uint64_t need = ns * h->G;
    if (words < need) return fail(BSRNG_EINVAL, "host buffer too small: need %llu words", (unsigned long long)need);
    DeviceGuard dg(h->dev);
    if (!dg.ok) return fail(BSRNG_ECUDA, "cudaSetDevice(%d) failed", h->dev);
    cudaError_t e = cudaDeviceSynchronize();
    if (e == cudaSuccess)
        e = cudaMemcpy2D(host_out, h->G * 4, h->state, h->Gp * 4, h->G * 4, ns, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "copy_state: %s", cudaGetErrorString(e));
    return int64_t(need);
}

int bsrng_set_option(bsrng_t* h, const char* key, int64_t value)
{
    if (!h || !key) return fail(BSRNG_EINVAL, "NULL argument");
    if (!strcmp(key, "sched")) {
        if (value != 0 && value != 1) return fail(BSRNG_EINVAL, "sched must be 0 or 1");
        h->opt_sched = int(value);
    } else if (!strcmp(key, "seg_clocks")) {
        if (value < 0 || value % 32) return fail(BSRNG_EINVAL, "seg_clocks must be a multiple of 32");
        h->opt_seg_clocks = uint64_t(value);
    } else if (!strcmp(key, "ctas_per_sm")) {
        if (value < 0 || value > 32) return fail(BSRNG_EINVAL, "ctas_per_sm out of range");
        h->opt_ctas_per_sm = int(value);
    } else if (!strcmp(key, "unroll")) {
        const bool grain = h->cipher == BSRNG_GRAIN_V1 || h->cipher == BSRNG_LFSR128;
        const bool ok = value == 0 || (grain ? (value == 8 || value == 16 || value == 32)
                                             : (value == 2 || value == 4 || value == 8));
        if (!ok) return fail(BSRNG_EINVAL, "unroll must be %s", grain ? "8, 16 or 32" : "2, 4 or 8");
        h->opt_unroll = int(value);
    } else if (!strcmp(key, "rm_ws")) {
        if (value < -1 || value > 1) return fail(BSRNG_EINVAL, "rm_ws must be -1 (auto), 0 or 1");
        h->opt_rm_ws = int(value);
    } else if (!strcmp(key, "rm_slots")) {
        if (value != 0 && value != 4 && value != 8) return fail(BSRNG_EINVAL, "rm_slots must be 0 (auto), 4 or 8");
        h->opt_rm_slots = int(value);
    } else if (!strcmp(key, "rm_zreg")) {
        if (value != 0 && value != 1) return fail(BSRNG_EINVAL, "rm_zreg must be 0 or 1");
        h->opt_rm_zreg = int(value);
    } else if (!strcmp(key, "rm_dbl")) {
        h->opt_rm_dbl = int(value);
    } else if (!strcmp(key, "rm_tma")) {
        h->opt_rm_tma = int(value);
    } else if (!strcmp(key, "rm_tmem")) {
        if (value < -1 || value > 1) return fail(BSRNG_EINVAL, "rm_tmem must be -1 (auto), 0 or 1");
        h->opt_rm_tmem = int(value);
    } else if (!strcmp(key, "init_fused")) {
        if (value != 0 && value != 1) return fail(BSRNG_EINVAL, "init_fused must be 0 or 1");
        h->opt_init_fused = int(value);
    } else if (!strcmp(key, "block")) {
        if (value != KS_BLOCK) return fail(BSRNG_EINVAL, "block=%lld not built (built: %d)", (long long)value, KS_BLOCK);
    } else {
        return fail(BSRNG_EINVAL, "unknown option '%s'", key);
    }
    return BSRNG_OK;
}

void bsrng_destroy(bsrng_t* h)
{
    if (!h) return;
    DeviceGuard dg(h->dev);
    if (h->state) cudaFree(h->state);
    if (h->sliced) cudaFree(h->sliced);
    if (h->raw) cudaFree(h->raw);
    if (h->sched) cudaFree(h->sched);
    if (h->bounce) cudaFree(h->bounce);
    if (h->rk_dev) cudaFree(h->rk_dev);
    if (h->tail) cudaFree(h->tail);
    delete h;
}

}  // extern "C"
