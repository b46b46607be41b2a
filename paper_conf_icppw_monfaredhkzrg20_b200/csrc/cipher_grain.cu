// cipher_grain.cu -- Grain v1 (sec. 2.3.3; spec [15]): the
// initialisation and keystream launches of libbsrng.so.
// Kernels: grain.cuh, keystream.cuh, rowmajor_ws.cuh; launcher: launch_ks.cuh.
#include "bitslice.cuh"
#include "grain.cuh"
#include "launch_ks.cuh"

namespace bsrng_impl {
namespace {

int init_grain(bsrng_t* h, cudaStream_t st, const uint8_t* raw_k, const uint8_t* raw_iv, uint64_t g_split)
{
    // spec [15]: key and IV bits are taken LSB-first from their bytes
    if (h->opt_init_fused) {
        if (int rc = set_smem(reinterpret_cast<const void*>(bsk::grain_init_kernel), bsk::GI_SMEM_BYTES)) return rc;
        bsk::grain_init_kernel<<<unsigned((h->Gp + GI_BLOCK - 1) / GI_BLOCK), GI_BLOCK, bsk::GI_SMEM_BYTES, st>>>(
            raw_k, raw_iv, h->tail, h->tail + h->tail_iv_off, g_split, h->state, h->Gp);
        return check_launch("grain_init");
    }
    if (g_split < h->Gp) return fail(BSRNG_EINVAL, "unfused init needs staged inputs");
    uint32_t* key_s = h->sliced;
    uint32_t* iv_s = h->sliced + 80 * h->Gp;
    const unsigned sblocks = unsigned((h->Gp + bsk::SLICE_GROUPS - 1) / bsk::SLICE_GROUPS);
    bsk::slice_bits_kernel<10, 80, false><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_k, h->n, key_s, h->Gp);
    if (int rc = check_launch("slice(key)")) return rc;
    bsk::slice_bits_kernel<8, 64, false><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_iv, h->n, iv_s, h->Gp);
    if (int rc = check_launch("slice(iv)")) return rc;
    bsk::grain_preclock_kernel<<<unsigned((h->Gp + 127) / 128), 128, 0, st>>>(key_s, iv_s, h->state, h->Gp);
    return check_launch("grain_preclock");
}

}  // namespace

const CipherOps k_grain_ops = {bsk::Grain::NSTATE, init_grain, generate_stream_cipher<bsk::Grain>};

}  // namespace bsrng_impl
