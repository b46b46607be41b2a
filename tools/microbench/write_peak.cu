// HBM write-only bandwidth on this B200 (context for the materialise paths,
// which only write): grid-stride streaming stores over a buffer much larger
// than L2, as 16 B (STG.128) and 4 B (STG.32: one 128 B line per warp
// instruction, the SLICED layout's pattern) stores, normal and evict-first.
// Plus the ROW_MAJOR flush pattern: warp w owns 32 rows of pitch P bytes and
// walks their columns in S-byte sectors (lane = row, S/16 16 B stores each),
// i.e. 32 rows P bytes apart per warp flush, as the materialise kernels write.
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

template <int S>
__global__ void __launch_bounds__(256) sector_kernel(void* p, size_t pitch, uint32_t seed)
{
    const size_t warp = (size_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
    const uint32_t lane = threadIdx.x & 31;
    uint4* row = reinterpret_cast<uint4*>(static_cast<char*>(p) + (warp * 32 + lane) * pitch);
    for (size_t c = 0; c < pitch / S; ++c) {
#pragma unroll
        for (int k = 0; k < S / 16; ++k)
            __stcs(row + c * (S / 16) + k, make_uint4(seed ^ uint32_t(c), lane, uint32_t(warp), k));
    }
}

// 32 B sectors with lane pairs per row (lane l: row l/2, half l%2): one store
// instruction writes 16 whole sectors, two instructions per 32-row flush
__global__ void __launch_bounds__(256) sector_pair_kernel(void* p, size_t pitch, uint32_t seed)
{
    const size_t warp = (size_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
    const uint32_t lane = threadIdx.x & 31;
    char* base = static_cast<char*>(p) + warp * 32 * pitch + (lane & 1) * 16;
    for (size_t c = 0; c < pitch / 32; ++c) {
#pragma unroll
        for (int h = 0; h < 2; ++h)
            __stcs(reinterpret_cast<uint4*>(base + (h * 16 + (lane >> 1)) * pitch + c * 32),
                   make_uint4(seed ^ uint32_t(c), lane, uint32_t(warp), h));
    }
}

template <int S>
void run_sector(void* buf, size_t nbytes, size_t pitch)
{
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    const size_t rows = nbytes / pitch;
    float best = 1e30f;
    for (int r = 0; r < 6; ++r) {
        cudaEventRecord(a);
        if constexpr (S == 0)
            sector_pair_kernel<<<unsigned(rows / 256), 256>>>(buf, pitch, 0x9E3779B9u + r);
        else
            sector_kernel<S><<<unsigned(rows / 256), 256>>>(buf, pitch, 0x9E3779B9u + r);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r > 0 && ms < best) best = ms;
    }
    if (S == 0)
        printf("{\"store\": \"row sectors 32 B as lane pairs (16 rows per STG.128), pitch %zu B, 32 rows per warp\", \"bytes\": %zu, \"ms\": %.3f, \"write_gbs\": %.1f}\n",
               pitch, rows * pitch, best, rows * pitch / (best * 1e-3) / 1e9);
    else
    printf("{\"store\": \"row sectors %d B, pitch %zu B, 32 rows per warp\", \"bytes\": %zu, \"ms\": %.3f, \"write_gbs\": %.1f}\n",
           S, pitch, rows * pitch, best, rows * pitch / (best * 1e-3) / 1e9);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
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
    for (size_t pitch : {size_t(4096), size_t(8192), size_t(65536)}) {
        run_sector<0>(buf, nbytes, pitch);
        run_sector<32>(buf, nbytes, pitch);
        run_sector<64>(buf, nbytes, pitch);
        run_sector<128>(buf, nbytes, pitch);
    }
    cudaFree(buf);
    return 0;
}
