// internal.h -- host-side internals shared by the translation units of
// libbsrng.so: the handle, error reporting, and the per-cipher entry points.
//
// The library is split per cipher (cipher_mickey2.cu, cipher_grain.cu,
// cipher_lfsr.cu, cipher_aes.cu) so the kernel instances compile in parallel;
// bsrng.cu holds the C ABI (include/bsrng.h) and dispatches through
// `CipherOps`.  Nothing here is visible outside the library.
#pragma once
#include <cuda.h>  // CUtensorMap (type only)
#include <cuda_runtime.h>

#include <cstdint>
#include <string>

#include "../../include/bsrng.h"

namespace bsrng_impl {

// printf-style failure: records the thread-local message, returns `code`
int fail(int code, const char* fmt, ...);
// counts a launch and converts a pending launch error into BSRNG_ECUDA
int check_launch(const char* what);
// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) for kernels above 48 KB.
// The attribute is per device, so it is set before every such launch (a
// process may hold handles on several GPUs).
int set_smem(const void* kern, size_t bytes);
// 3-D TMA view [q 32][group][byte] of a ROW_MAJOR output (keystream.cuh)
int encode_rowmajor_tmap(CUtensorMap* map, void* out, uint64_t row_bytes, uint64_t groups);

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

// Longest work item (clocks) of one keystream launch: the kernels count an
// item's clocks in 32 bits, so longer calls are split into time segments.
constexpr uint64_t MAX_SEG_CLOCKS = 1ull << 31;

}  // namespace bsrng_impl

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
    uint32_t* sliced = nullptr;  // key [KB][Gp] then iv [IVB][Gp] (unfused init only)
    uint8_t* raw = nullptr;      // keys [Gp*32][key_bytes] then ivs at raw + iv_off (zero-padded)
    uint64_t iv_off = 0;         // per-instance regions padded to Gp*32 rows (zeroed), 16 B aligned
    uint32_t* sched = nullptr;   // [1 + units]: ticket, flags; then [32] scratch; then [1] second ticket
    // AES ROW_MAJOR: the instance-sliced remainder kernel runs on this side
    // stream beside the block-lane kernel (fork / join events on the caller's stream)
    cudaStream_t side = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    uint8_t* bounce = nullptr;   // generate_host staging
    uint64_t bounce_bytes = 0;
    // host inputs are copied into this handle-owned pinned buffer before the
    // asynchronous H2D copy, so the caller may reuse its buffers on return
    uint8_t* pinned = nullptr;
    uint64_t pinned_bytes = 0;
    cudaEvent_t pinned_free = nullptr;  // recorded after the last H2D copy out of `pinned`
    // device-input rekeys read whole 32-instance groups straight from the
    // caller's arrays; the partial last group and the padding groups (< 32)
    // come from this zeroed buffer: keys [32 groups * 32][key_bytes], then IVs
    uint8_t* tail = nullptr;
    uint64_t tail_iv_off = 0;
    // AES: round-key masks written by the key-expansion kernel, then copied
    // (device to device, stream-ordered) into constant-memory slot `aes_slot`
    uint32_t* rk_dev = nullptr;
    int aes_slot = -1;
    // options
    int opt_sched = 1;
    uint64_t opt_seg_clocks = 0;
    int opt_ctas_per_sm = 0;  // resident CTAs per SM; 0 = auto
    int opt_unroll = 0;       // 0 = the cipher's default (MICKEY 4, Grain/LFSR 32)
    // ROW_MAJOR kernel: -1 auto, 1 warp-specialised (AES: block-lane), 0 plain
    int opt_rm_ws = -1;
    // ROW_MAJOR plain kernel: stage row segments in TMEM (1) or smem (0); -1 = cipher default
    int opt_rm_tmem = -1;
    // TMEM-staged ROW_MAJOR: whole-sector flushes as TMA tensor stores (1) or 8 B stores (0)
    int opt_rm_tma = 1;
    // TMEM-staged ROW_MAJOR with one CTA per SM: double-buffered staging (1) or not (0)
    int opt_rm_dbl = 1;
    // ROW_MAJOR: 64 B TMEM staging per row, one clock-loop warp per SMSP (1)
    int opt_rm_wide = 0;
    // ROW_MAJOR 32 B flushes with an L2 evict_last hint (1, default: a row's
    // next sector then finds its 128 B line resident; Grain C2 11.5 vs 10.5
    // Tb/s) or evict-first (0)
    int opt_rm_l2last = 1;
    // writer-warp kernel: staggered 64 B flush periods per warp-unit (-1 auto:
    // on when rows are not 16 B aligned, e.g. the paper's 552 B rows)
    int opt_rm_phase = -1;
    // init: slicing fused into the init kernel (1) or the ballot slice kernels (0)
    int opt_init_fused = 1;
};

namespace bsrng_impl {

// Per-cipher entry points (cipher_*.cu).
//   init    : slice + initialisation clocks into h->state from group blocks
//             raw_k / raw_iv (+ g * 32 * bytes) for groups g < g_split, the
//             rest from h->tail (the staged path passes h->raw, g_split = Gp)
//   generate: one bsrng_generate call (arguments validated by the caller)
struct CipherOps {
    int nstate;
    int (*init)(bsrng_t* h, cudaStream_t st, const uint8_t* raw_k, const uint8_t* raw_iv, uint64_t g_split);
    int (*generate)(bsrng_t* h, void* out, uint64_t bits, bsrng_layout layout, cudaStream_t st);
};
extern const CipherOps k_mickey2_ops, k_grain_ops, k_lfsr_ops, k_aes_ops;

// AES-128-CTR constant-memory round-key slots (cipher_aes.cu)
int aes_acquire_slot();
void aes_release_slot(int slot);

}  // namespace bsrng_impl
