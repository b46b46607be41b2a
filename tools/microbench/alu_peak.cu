// alu_peak.cu -- measure the B200 integer-logic (LOP3) issue ceiling that the
// MICKEY roofline is quoted against.
//
// Each thread runs CH independent lop3.b32 dependency chains for ITERS
// iterations; the grid fills every SM with W warps.  Variants add IMAD.MOV-class
// work (FMA pipe) to check whether it co-issues with the ALU pipe.
//   build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o alu_peak alu_peak.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

template <int LUT>
__device__ __forceinline__ unsigned lop3(unsigned a, unsigned b, unsigned c)
{
    unsigned d;
    asm volatile("lop3.b32 %0, %1, %2, %3, %4;" : "=r"(d) : "r"(a), "r"(b), "r"(c), "n"(LUT));
    return d;
}

template <int CH, int FMA_PER_8>
__global__ void lop3_kernel(unsigned* out, int iters, unsigned seed)
{
    unsigned x[CH];
    unsigned k1 = seed * 0x9E3779B9u + threadIdx.x, k2 = seed ^ blockIdx.x;
#pragma unroll
    for (int i = 0; i < CH; ++i) x[i] = seed + i * 77u + threadIdx.x;
    float f0 = __uint_as_float(k1 & 0x3fffffff), f1 = 1.0001f;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 8; ++r) {
#pragma unroll
            for (int i = 0; i < CH; ++i) x[i] = lop3<0x96>(x[i], k1, k2 + r);
#pragma unroll
            for (int j = 0; j < FMA_PER_8; ++j) f0 = fmaf(f0, f1, 1.0f);
        }
    }
    unsigned acc = 0;
#pragma unroll
    for (int i = 0; i < CH; ++i) acc ^= x[i];
    if (acc == 0x12345678u && f0 == 0.0f) out[0] = acc;
}

template <int CH, int F>
void run(const char* name, int sms, int warps_per_sm, int iters)
{
    unsigned* d;
    cudaMalloc(&d, 4);
    dim3 grid(sms * warps_per_sm / 4), block(128);
    lop3_kernel<CH, F><<<grid, block>>>(d, iters / 8, 1);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventRecord(e0);
    lop3_kernel<CH, F><<<grid, block>>>(d, iters, 1);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double ops = double(grid.x) * block.x * iters * 8.0 * CH;
    int clk_khz;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    printf("{\"variant\": \"%s\", \"warps_per_sm\": %d, \"chains\": %d, \"fma_per_8_lop3\": %d, \"ms\": %.3f, "
           "\"tlop3_per_s\": %.3f, \"lop3_per_clk_per_sm_at_attr_clock\": %.2f, \"attr_clock_mhz\": %d}\n",
           name, warps_per_sm, CH, F, ms, ops / (ms * 1e-3) / 1e12, ops / (ms * 1e-3) / (clk_khz * 1e3) / sms,
           clk_khz / 1000);
    cudaFree(d);
}

int main(int argc, char** argv)
{
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int iters = argc > 1 ? atoi(argv[1]) : 200000;
    run<8, 0>("lop3", sms, 4, iters);
    run<8, 0>("lop3", sms, 8, iters);
    run<8, 0>("lop3", sms, 16, iters);
    run<4, 0>("lop3", sms, 16, iters);
    run<8, 4>("lop3+ffma", sms, 8, iters);
    run<8, 8>("lop3+ffma", sms, 8, iters);
    return 0;
}
