// HBM write-only bandwidth on this B200 (context for the materialise paths,
// which only write): grid-stride streaming stores over a buffer much larger
// than L2, as 16 B (STG.128) and 4 B (STG.32: one 128 B line per warp
// instruction, the SLICED layout's pattern) stores, normal and evict-first.
// Prints one JSON line per variant: best of 5 launches, CUDA events.
#include <cstdint>
#include <cstdio>

template <int W, bool CS>
__global__ void __launch_bounds__(256) write_kernel(void* p, size_t nbytes, uint32_t seed)
{
    const size_t n = nbytes / (W == 16 ? 16 : 4);
    size_t i = size_t(blockIdx.x) * blockDim.x + threadIdx.x;
    const size_t stride = size_t(gridDim.x) * blockDim.x;
    if constexpr (W == 16) {
        uint4* q = static_cast<uint4*>(p);
        for (; i < n; i += stride) {
            const uint4 v = make_uint4(seed ^ uint32_t(i), seed, uint32_t(i >> 32), seed + 1);
            if (CS) __stcs(q + i, v); else q[i] = v;
        }
    } else {
        uint32_t* q = static_cast<uint32_t*>(p);
        for (; i < n; i += stride) {
            if (CS) __stcs(q + i, seed ^ uint32_t(i)); else q[i] = seed ^ uint32_t(i);
        }
    }
}

template <int W, bool CS>
void run(void* buf, size_t nbytes, int sms)
{
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int r = 0; r < 6; ++r) {
        cudaEventRecord(a);
        write_kernel<W, CS><<<sms * 8, 256>>>(buf, nbytes, 0x9E3779B9u + r);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r > 0 && ms < best) best = ms;
    }
    printf("{\"store\": \"STG.%d%s\", \"bytes\": %zu, \"ms\": %.3f, \"write_gbs\": %.1f}\n", W * 8,
           CS ? " evict-first" : "", nbytes, best, nbytes / (best * 1e-3) / 1e9);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
}

int main()
{
    const size_t nbytes = size_t(8) << 30;
    void* buf;
    if (cudaMalloc(&buf, nbytes) != cudaSuccess) { printf("{\"error\": \"cudaMalloc\"}\n"); return 1; }
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    run<16, false>(buf, nbytes, sms);
    run<16, true>(buf, nbytes, sms);
    run<4, false>(buf, nbytes, sms);
    run<4, true>(buf, nbytes, sms);
    cudaFree(buf);
    return 0;
}
