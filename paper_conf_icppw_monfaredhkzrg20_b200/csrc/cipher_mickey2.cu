// cipher_mickey2.cu -- MICKEY 2.0 (sec. 2.3.1, sec. 4.4; spec
// [5]): the initialisation (SURVEY steps a-1 + a-2) and keystream (a-3..a-5)
// launches of libbsrng.so.  Kernels: mickey2.cuh, keystream.cuh,
// rowmajor_ws.cuh; launcher: launch_ks.cuh.
#include "bitslice.cuh"
#include "launch_ks.cuh"
#include "mickey2.cuh"

namespace bsrng_impl {
namespace {

int init_mickey2(bsrng_t* h, cudaStream_t st, const uint8_t* raw_k, const uint8_t* raw_iv, uint64_t g_split)
{
    if (h->opt_init_fused) {
        // one kernel: slicing in registers/shared memory + the iv_bits + 180 mixing clocks
        const unsigned blocks = unsigned((h->Gp + bsk::M2I_BLOCK - 1) / bsk::M2I_BLOCK);
        if (int rc = set_smem(reinterpret_cast<const void*>(bsk::m2_init_kernel), bsk::M2I_SMEM_BYTES)) return rc;
        bsk::m2_init_kernel<<<blocks, bsk::M2I_BLOCK, bsk::M2I_SMEM_BYTES, st>>>(
            raw_k, raw_iv, h->tail, h->tail + h->tail_iv_off, g_split, int(h->iv_bits), h->state, h->Gp);
        return check_launch("m2_init");
    }
    if (g_split < h->Gp) return fail(BSRNG_EINVAL, "unfused init needs staged inputs");
    uint32_t* key_s = h->sliced;
    uint32_t* iv_s = h->sliced + 80 * h->Gp;
    const unsigned sblocks = unsigned((h->Gp + bsk::SLICE_GROUPS - 1) / bsk::SLICE_GROUPS);
    bsk::slice_bits_kernel<10, 80, true><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_k, h->n, key_s, h->Gp);
    if (int rc = check_launch("slice(key)")) return rc;
    bsk::slice_bits_kernel<10, 80, true><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_iv, h->n, iv_s, h->Gp);
    if (int rc = check_launch("slice(iv)")) return rc;
    bsk::m2_preclock_kernel<<<unsigned((h->Gp + 127) / 128), 128, 0, st>>>(iv_s, key_s, int(h->iv_bits), h->state,
                                                                          h->Gp);
    return check_launch("m2_preclock");
}

}  // namespace

const CipherOps k_mickey2_ops = {bsk::Mickey2::NSTATE, init_mickey2, generate_stream_cipher<bsk::Mickey2>};

}  // namespace bsrng_impl
