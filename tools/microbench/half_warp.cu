// half_warp.cu -- does a warp with only 16 active lanes issue LOP3 at twice the
// rate of a full warp on the B200's 16-lane-per-SMSP integer pipe?  (Would let
// the paper shape's 512 warp-units run as 1024 half-warps, two per SMSP.)
//   build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o half_warp half_warp.cu
#include <cstdio>
#include <cuda_runtime.h>

template <int LUT>
__device__ __forceinline__ unsigned lop3(unsigned a, unsigned b, unsigned c)
{
    unsigned d;
    asm volatile("lop3.b32 %0, %1, %2, %3, %4;" : "=r"(d) : "r"(a), "r"(b), "r"(c), "n"(LUT));
    return d;
}

template <int CH>
__global__ void k(unsigned* out, int iters, int active)
{
    if ((threadIdx.x & 31) >= unsigned(active)) return;
    unsigned x[CH];
    unsigned k1 = threadIdx.x * 0x9E3779B9u, k2 = blockIdx.x;
#pragma unroll
    for (int i = 0; i < CH; ++i) x[i] = i * 77u + threadIdx.x;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 8; ++r) {
#pragma unroll
            for (int i = 0; i < CH; ++i) x[i] = lop3<0x96>(x[i], k1, k2 + r);
        }
    }
    unsigned acc = 0;
#pragma unroll
    for (int i = 0; i < CH; ++i) acc ^= x[i];
    if (acc == 0x12345678u) out[0] = acc;
}

int main()
{
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    unsigned* d;
    cudaMalloc(&d, 4);
    const int iters = 100000;
    for (int wps : {4, 8}) {
        for (int active : {32, 16, 8}) {
            dim3 grid(sms * wps / 4), block(128);
            k<8><<<grid, block>>>(d, iters / 10, active);
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0);
            cudaEventCreate(&e1);
            cudaEventRecord(e0);
            k<8><<<grid, block>>>(d, iters, active);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            const double warp_instr = double(grid.x) * 4 * iters * 8.0 * 8;
            printf("warps/SM %d active lanes %2d: %.3f ms, %.3f warp-LOP3 per clk per SMSP (at 1965 MHz)\n", wps,
                   active, ms, warp_instr / (ms * 1e-3) / 1965e6 / (sms * 4));
        }
    }
    return 0;
}
