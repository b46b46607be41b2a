// cipher_lfsr.cu -- the paper's bitsliced LFSR (sec. 4.3, Eq.
// 2): key slicing (the sliced key IS the state) and keystream
// launches of libbsrng.so.  Kernels: lfsr.cuh, keystream.cuh; launcher:
// launch_ks.cuh.
#include "bitslice.cuh"
#include "launch_ks.cuh"
#include "lfsr.cuh"

namespace bsrng_impl {
namespace {

int init_lfsr(bsrng_t* h, cudaStream_t st, const uint8_t* raw_k, const uint8_t*, uint64_t g_split)
{
    // the state IS the key: 128 bits, MSB-first, sliced straight into rows 0..127
    if (h->opt_init_fused) {
        if (int rc = set_smem(reinterpret_cast<const void*>(bsk::slice_state_kernel<16, 128, true>),
                              bsk::ss_smem_bytes(16)))
            return rc;
        bsk::slice_state_kernel<16, 128, true><<<unsigned((h->Gp + 127) / 128), 128, bsk::ss_smem_bytes(16), st>>>(
            raw_k, h->tail, g_split, h->state, h->Gp);
    } else if (g_split >= h->Gp) {
        const unsigned sblocks = unsigned((h->Gp + bsk::SLICE_GROUPS - 1) / bsk::SLICE_GROUPS);
        bsk::slice_bits_kernel<16, 128, true><<<sblocks, bsk::SLICE_BLOCK, 0, st>>>(raw_k, h->n, h->state, h->Gp);
    } else {
        return fail(BSRNG_EINVAL, "unfused init needs staged inputs");
    }
    if (int rc = check_launch("slice(key)")) return rc;
    cudaError_t e = cudaMemsetAsync(h->state + uint64_t(bsk::Lfsr128::NSTATE) * h->Gp, 0, h->Gp * 4, st);
    if (e != cudaSuccess) return fail(BSRNG_ECUDA, "memset: %s", cudaGetErrorString(e));
    return BSRNG_OK;
}

}  // namespace

const CipherOps k_lfsr_ops = {bsk::Lfsr128::NSTATE, init_lfsr, generate_stream_cipher<bsk::Lfsr128>};

}  // namespace bsrng_impl
