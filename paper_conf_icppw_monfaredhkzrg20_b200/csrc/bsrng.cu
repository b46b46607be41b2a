// bsrng.cu -- host side of the C ABI declared in include/bsrng.h.
//
// Handle = device-resident sliced cipher state [NSTATE + 1][Gp] (HBM) plus
// scratch for key/IV slicing and the persistent scheduler.  Every entry point
// validates its arguments, switches to the handle's device, enqueues kernels on
// the caller's stream and reports errors through a thread-local string.  The
// kernels are launched by the per-cipher translation units (cipher_*.cu,
// internal.h).  There is no CPU fallback anywhere in this library.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>

#include "internal.h"

namespace bsrng_impl {

namespace {
thread_local std::string g_err;
std::atomic<uint64_t> g_launches{0};
}  // namespace

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

int check_launch(const char* what)
{
    g_launches.fetch_add(1, std::memory_order_relaxed);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "%s launch failed: %s", what, cudaGetErrorString(e));
    return BSRNG_OK;
}

int set_smem(const void* kern, size_t bytes)
{
    if (bytes <= 48 * 1024) return BSRNG_OK;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(bytes));
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "smem attribute (%zu B): %s", bytes, cudaGetErrorString(e));
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
    static std::atomic<EncodeTiledFn> encode{nullptr};
    EncodeTiledFn fn_ptr = encode.load();
    if (!fn_ptr) {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess || !fn)
            return fail(BSRNG_ECUDA, "cuTensorMapEncodeTiled unavailable");
        fn_ptr = reinterpret_cast<EncodeTiledFn>(fn);
        encode.store(fn_ptr);
    }
    const cuuint64_t dims[3] = {row_bytes, groups, 32};
    const cuuint64_t strides[2] = {32 * row_bytes, row_bytes};
    const cuuint32_t box[3] = {32, 8, 32}, estr[3] = {1, 1, 1};
    const CUresult r = fn_ptr(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, out, dims, strides, box, estr,
                              CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                              CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return fail(BSRNG_ECUDA, "cuTensorMapEncodeTiled failed (%d)", int(r));
    return BSRNG_OK;
}

}  // namespace bsrng_impl

using namespace bsrng_impl;

namespace {

const CipherOps* ops_of(bsrng_cipher c)
{
    switch (c) {
    case BSRNG_MICKEY2: return &k_mickey2_ops;
    case BSRNG_GRAIN_V1: return &k_grain_ops;
    case BSRNG_AES128_CTR: return &k_aes_ops;
    case BSRNG_LFSR128: return &k_lfsr_ops;
    default: return nullptr;
    }
}

// keystream bits per key/IV: MICKEY 2.0's limit is 2^40;
// Grain, AES-CTR and the LFSR are only bounded by the 64-bit bit counter here.
uint64_t max_bits(bsrng_cipher c) { return c == BSRNG_MICKEY2 ? (1ull << 40) : (1ull << 62); }

// EINVAL unless `stream` belongs to the handle's device (call under DeviceGuard:
// the NULL / legacy / per-thread streams then resolve to that device).
int check_stream(const bsrng_t* h, cudaStream_t st)
{
    // NULL and the special legacy / per-thread handles name the current
    // device's stream, which the caller's DeviceGuard made the handle's
    if (!st || st == cudaStreamLegacy || st == cudaStreamPerThread) return BSRNG_OK;
    int sdev = -1;
    cudaError_t e = cudaStreamGetDevice(st, &sdev);
    if (e != cudaSuccess) {
        cudaGetLastError();
        return fail(BSRNG_EINVAL, "invalid stream: %s", cudaGetErrorString(e));
    }
    if (sdev != h->dev) return fail(BSRNG_EINVAL, "stream belongs to device %d, the handle to device %d", sdev, h->dev);
    return BSRNG_OK;
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

// Host inputs: copied into the handle-owned pinned buffer (after the previous
// H2D copy out of it has completed), then H2D-copied asynchronously from
// there, so the caller may overwrite its buffers as soon as the call returns.
int stage_host_inputs(bsrng_t* h, const uint8_t* keys, const uint8_t* ivs, cudaStream_t st)
{
    const uint64_t kb = h->key_rows * h->key_bytes, vb = ivs ? h->n * h->iv_bytes : 0;
    if (h->pinned_bytes < kb + vb) {
        if (h->pinned_free) cudaEventSynchronize(h->pinned_free);
        if (h->pinned) cudaFreeHost(h->pinned);
        h->pinned = nullptr;
        h->pinned_bytes = 0;
        if (cudaMallocHost(&h->pinned, kb + vb) != cudaSuccess) {
            cudaGetLastError();
            return fail(BSRNG_ENOMEM, "cudaMallocHost(%llu) for input staging", (unsigned long long)(kb + vb));
        }
        h->pinned_bytes = kb + vb;
    }
    if (!h->pinned_free && cudaEventCreateWithFlags(&h->pinned_free, cudaEventDisableTiming) != cudaSuccess)
        return fail(BSRNG_ECUDA, "cudaEventCreate failed");
    cudaError_t e = cudaEventSynchronize(h->pinned_free);  // previous copy out of the buffer done
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "staging wait: %s", cudaGetErrorString(e));
    memcpy(h->pinned, keys, kb);
    if (vb) memcpy(h->pinned + kb, ivs, vb);
    e = cudaMemcpyAsync(h->raw, h->pinned, kb, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess && vb) e = cudaMemcpyAsync(h->raw + h->iv_off, h->pinned + kb, vb, cudaMemcpyHostToDevice, st);
    if (e == cudaSuccess) e = cudaEventRecord(h->pinned_free, st);
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "key/iv copy failed: %s", cudaGetErrorString(e));
    return BSRNG_OK;
}

}  // namespace

extern "C" {

const char* bsrng_last_error(void) { return bsrng_impl::g_err.c_str(); }

uint64_t bsrng_launch_count(void) { return bsrng_impl::g_launches.load(); }

bsrng_t* bsrng_create_ex(bsrng_cipher cipher, const uint8_t* keys, const uint8_t* ivs, uint32_t iv_bits,
                         uint64_t n, uint64_t first_instance_id, uint32_t flags, void* stream)
{
    g_err.clear();
    const CipherOps* ops = ops_of(cipher);
    if (!ops) {
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
    if (cipher == BSRNG_MICKEY2 && iv_bits > 80) {
        fail(BSRNG_EINVAL, "MICKEY iv_bits=%u must be in [0, 80]", iv_bits);
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
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (check_stream(h, st) != BSRNG_OK) {
        std::string msg = g_err;
        delete h;
        g_err = msg;
        return nullptr;
    }
    const bool aes = cipher == BSRNG_AES128_CTR, lfsr = cipher == BSRNG_LFSR128;
    h->key_bytes = (aes || lfsr) ? 16 : 10;
    h->iv_bytes = cipher == BSRNG_GRAIN_V1 ? 8 : aes ? 16 : lfsr ? 0 : 10;
    h->key_rows = aes ? 1 : h->n;
    if (aes && (h->aes_slot = aes_acquire_slot()) < 0) {
        delete h;
        fail(BSRNG_ENOMEM, "all %d AES-128-CTR round-key slots are in use (one per live AES handle)", 11);
        return nullptr;
    }
    // the fused init kernels read whole 32-instance group blocks with 16 B
    // loads: the per-instance regions are padded to Gp*32 rows and zeroed
    h->iv_off = aes ? 16 : h->Gp * 32 * h->key_bytes;  // AES: one 16 B key
    const uint64_t raw_bytes = h->iv_off + h->Gp * 32 * h->iv_bytes;
    const uint64_t sl_words = (aes || lfsr) ? 1 : uint64_t(h->key_bytes + h->iv_bytes) * 8 * h->Gp;
    if (cudaMalloc(&h->state, uint64_t(ops->nstate + 1) * h->Gp * 4) != cudaSuccess ||
        cudaMalloc(&h->sliced, sl_words * 4) != cudaSuccess ||
        cudaMalloc(&h->raw, raw_bytes) != cudaSuccess ||
        cudaMalloc(&h->sched, (1 + h->units + 32 + 1) * 4) != cudaSuccess ||
        (aes && cudaMalloc(&h->rk_dev, 11 * 128 * 4) != cudaSuccess) ||
        cudaMalloc(&h->tail, 32 * 32 * uint64_t(h->key_bytes + h->iv_bytes)) != cudaSuccess) {
        cudaGetLastError();
        bsrng_destroy(h);
        fail(BSRNG_ENOMEM, "cudaMalloc failed for %llu instances", (unsigned long long)n);
        return nullptr;
    }
    h->tail_iv_off = 32 * 32 * uint64_t(h->key_bytes);
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
    if (flags & ~uint32_t(BSRNG_INPUT_DEVICE)) return fail(BSRNG_EINVAL, "unknown flags 0x%x", flags);
    DeviceGuard dg(h->dev);
    if (!dg.ok) return fail(BSRNG_ECUDA, "cudaSetDevice(%d) failed", h->dev);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (int rc = check_stream(h, st)) return rc;
    const CipherOps* ops = ops_of(h->cipher);
    const bool aes = h->cipher == BSRNG_AES128_CTR;
    // Device inputs, 16 B aligned, fused init: the init kernels read whole
    // groups straight from the caller's arrays (no staging copy, ~25 us per
    // 2^22 keys); only the partial last group goes through h->tail.
    const bool direct = (flags & BSRNG_INPUT_DEVICE) && h->opt_init_fused && ivs &&
                        ((reinterpret_cast<uintptr_t>(keys) | reinterpret_cast<uintptr_t>(ivs)) & 15) == 0;
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
        if (int rc = ops->init(h, st, keys, ivs, g_split)) return rc;
        h->bits_done = 0;
        return BSRNG_OK;
    }
    if (!ivs && h->iv_bytes) {  // iv_bits == 0: IV bytes are never read; keep them defined
        cudaError_t e = cudaMemsetAsync(h->raw + h->iv_off, 0, h->n * h->iv_bytes, st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset: %s", cudaGetErrorString(e));
    }
    if (flags & BSRNG_INPUT_DEVICE) {
        cudaError_t e = cudaMemcpyAsync(h->raw, keys, h->key_rows * h->key_bytes, cudaMemcpyDeviceToDevice, st);
        if (e == cudaSuccess && ivs && h->iv_bytes)
            e = cudaMemcpyAsync(h->raw + h->iv_off, ivs, h->n * h->iv_bytes, cudaMemcpyDeviceToDevice, st);
        if (e != cudaSuccess) return fail(BSRNG_ECUDA, "key/iv copy failed: %s", cudaGetErrorString(e));
    } else if (int rc = stage_host_inputs(h, keys, h->iv_bytes ? ivs : nullptr, st)) {
        return rc;
    }
    if (int rc = ops->init(h, st, h->raw, h->raw + h->iv_off, h->Gp)) return rc;
    h->bits_done = 0;
    return BSRNG_OK;
}

int bsrng_generate(bsrng_t* h, void* out, uint64_t bits, bsrng_layout layout, void* stream)
{
    if (int rc = validate_generate(h, out, bits, layout, false)) return rc;
    DeviceGuard dg(h->dev);
    if (!dg.ok) return fail(BSRNG_ECUDA, "cudaSetDevice(%d) failed", h->dev);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (int rc = check_stream(h, st)) return rc;
    if (bits == 0) return BSRNG_OK;
    const int rc = ops_of(h->cipher)->generate(h, out, bits, layout, st);
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
    DeviceGuard dg(h->dev);
    if (!dg.ok) return fail(BSRNG_ECUDA, "cudaSetDevice(%d) failed", h->dev);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    if (int rc = check_stream(h, st)) return rc;
    if (bits == 0) return BSRNG_OK;
    // chunk so the device staging buffer stays <= 1 GiB
    const uint64_t cap = 1ull << 30;
    uint64_t per_clock = layout == BSRNG_ROW_MAJOR ? (h->n + 7) / 8 : layout == BSRNG_SLICED ? h->G * 4 : 0;
    uint64_t chunk = bits;
    const uint64_t cq = h->cipher == BSRNG_AES128_CTR ? 256 : 32;
    if (per_clock) chunk = std::max<uint64_t>(cq, std::min<uint64_t>(bits, cap / per_clock / cq * cq));
    if (layout == BSRNG_CHECKSUM) chunk = bits;  // a checksum covers the whole call
    const uint64_t need = bsrng_out_bytes(h, chunk, layout);
    if (h->bounce_bytes < need) {
        if (h->bounce) {
            cudaStreamSynchronize(st);
            cudaFree(h->bounce);
        }
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
    const uint64_t ns = uint64_t(ops_of(h->cipher)->nstate);
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
    auto in01 = [&](const char* what) { return (value == 0 || value == 1) ? BSRNG_OK : fail(BSRNG_EINVAL, "%s must be 0 or 1", what); };
    if (!strcmp(key, "sched")) {
        if (int rc = in01("sched")) return rc;
        h->opt_sched = int(value);
    } else if (!strcmp(key, "seg_clocks")) {
        if (value < 0 || value % 32) return fail(BSRNG_EINVAL, "seg_clocks must be a non-negative multiple of 32");
        h->opt_seg_clocks = uint64_t(value);
    } else if (!strcmp(key, "ctas_per_sm")) {
        if (value < 0 || value > 32) return fail(BSRNG_EINVAL, "ctas_per_sm out of range");
        h->opt_ctas_per_sm = int(value);
    } else if (!strcmp(key, "unroll")) {
        const bool wide = h->cipher == BSRNG_GRAIN_V1 || h->cipher == BSRNG_LFSR128;
        // built unrolls: Grain / LFSR 32 (default) and 16, MICKEY 4; AES has none
        const bool ok = value == 0 || (wide ? (value == 16 || value == 32) : h->cipher == BSRNG_MICKEY2 && value == 4);
        if (!ok) return fail(BSRNG_EINVAL, "unroll must be %s", wide ? "16 or 32" : "4 (MICKEY; AES: none)");
        h->opt_unroll = int(value);
    } else if (!strcmp(key, "rm_ws")) {
        if (value < -1 || value > 2) return fail(BSRNG_EINVAL, "rm_ws must be -1 (auto), 0, 1 or 2");
        h->opt_rm_ws = int(value);
    } else if (!strcmp(key, "rm_dbl")) {
        if (int rc = in01("rm_dbl")) return rc;
        h->opt_rm_dbl = int(value);
    } else if (!strcmp(key, "rm_tma")) {
        if (int rc = in01("rm_tma")) return rc;
        h->opt_rm_tma = int(value);
    } else if (!strcmp(key, "rm_wide")) {
        if (int rc = in01("rm_wide")) return rc;
        h->opt_rm_wide = int(value);
    } else if (!strcmp(key, "rm_l2last")) {
        if (int rc = in01("rm_l2last")) return rc;
        h->opt_rm_l2last = int(value);
    } else if (!strcmp(key, "rm_phase")) {
        if (value < -1 || value > 1) return fail(BSRNG_EINVAL, "rm_phase must be -1 (auto), 0 or 1");
        h->opt_rm_phase = int(value);
    } else if (!strcmp(key, "rm_tmem")) {
        if (value < -1 || value > 1) return fail(BSRNG_EINVAL, "rm_tmem must be -1 (auto), 0 or 1");
        h->opt_rm_tmem = int(value);
    } else if (!strcmp(key, "init_fused")) {
        if (int rc = in01("init_fused")) return rc;
        h->opt_init_fused = int(value);
    } else {
        return fail(BSRNG_EINVAL, "unknown option '%s'", key);
    }
    return BSRNG_OK;
}

void bsrng_destroy(bsrng_t* h)
{
    if (!h) return;
    DeviceGuard dg(h->dev);
    if (h->pinned_free) {
        cudaEventSynchronize(h->pinned_free);
        cudaEventDestroy(h->pinned_free);
    }
    if (h->pinned) cudaFreeHost(h->pinned);
    if (h->state) cudaFree(h->state);
    if (h->sliced) cudaFree(h->sliced);
    if (h->raw) cudaFree(h->raw);
    if (h->sched) cudaFree(h->sched);
    if (h->side) {
        cudaStreamSynchronize(h->side);
        cudaStreamDestroy(h->side);
    }
    if (h->ev_fork) cudaEventDestroy(h->ev_fork);
    if (h->ev_join) cudaEventDestroy(h->ev_join);
    if (h->bounce) cudaFree(h->bounce);
    if (h->rk_dev) cudaFree(h->rk_dev);
    if (h->tail) cudaFree(h->tail);
    aes_release_slot(h->aes_slot);
    delete h;
}

}  // extern "C"
