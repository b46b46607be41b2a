// grain_split_probe.cu -- feasibility probe for splitting one Grain v1 unit
// over two warps: how fast does a lone warp run the NFSR
// half alone (g + h + the b register, 34 LOP3 per clock) when the LFSR words
// it taps (s_t, s_t+3, s_t+25, s_t+46, s_t+64) come from a shared-memory ring?
// Compared with the whole cipher in a lone warp (~85 cycles per clock).
// One CTA of 4 warps per SM (one warp per SMSP), CUDA events, prints cycles
// per clock per warp at the sampled SM clock (pass it as argv[1], MHz).
#include <cstdint>
#include <cstdio>
#include <cstdlib>

template <uint32_t LUT>
__device__ __forceinline__ uint32_t lop3(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm("lop3.b32 %0, %1, %2, %3, %4;" : "=r"(d) : "r"(a), "r"(b), "r"(c), "n"(LUT));
    return d;
}
constexpr uint32_t XOR3 = 0x96u, XOR2 = 0x3Cu, AND3 = 0x80u, AND2 = 0xC0u, XAND = 0x78u, MUX = 0xCAu;

template <bool FULL>
__global__ void __launch_bounds__(128, 1) probe(uint32_t* out, int iters, uint32_t seed)
{
    extern __shared__ uint32_t ring_raw[];  // LFSR words, [index mod 256][thread] (128 KB, dynamic)
    uint32_t(*ring)[128] = reinterpret_cast<uint32_t(*)[128]>(ring_raw);
    const uint32_t tid = threadIdx.x;
    for (int i = 0; i < 256; ++i) ring[i][tid] = seed * (i + 1) ^ tid;
    __syncthreads();
    uint32_t b[80], s[80];
#pragma unroll
    for (int i = 0; i < 80; ++i) b[i] = seed ^ (i * 0x9E3779B9u) ^ tid, s[i] = b[i] * 3u;
    uint32_t acc = 0;
    uint32_t base = 0;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int u = 0; u < 32; ++u) {
            uint32_t s0, s3, s25, s46, s64;
            if (FULL) {
                s0 = s[0], s3 = s[3], s25 = s[25], s46 = s[46], s64 = s[64];
            } else {
                const uint32_t t = (base + u) & 255u;
                s0 = ring[t][tid];
                s3 = ring[(t + 3) & 255u][tid];
                s25 = ring[(t + 25) & 255u][tid];
                s46 = ring[(t + 46) & 255u][tid];
                s64 = ring[(t + 64) & 255u][tid];
            }
            // g (25)
            const uint32_t t1 = lop3<XOR3>(s0, b[62], b[60]);
            const uint32_t t2 = lop3<XOR3>(b[52], b[45], b[37]);
            const uint32_t t3 = lop3<XOR3>(b[33], b[28], b[21]);
            const uint32_t t4 = lop3<XOR3>(b[14], b[9], b[0]);
            const uint32_t q45 = lop3<AND2>(b[52], b[45], 0u);
            const uint32_t q21 = lop3<AND2>(b[28], b[21], 0u);
            const uint32_t p1 = lop3<AND2>(b[63], b[60], 0u);
            const uint32_t p2 = lop3<AND2>(b[37], b[33], 0u);
            const uint32_t p3 = lop3<AND2>(b[15], b[9], 0u);
            const uint32_t a1 = lop3<XAND>(t2, b[60], q45);
            const uint32_t p5 = lop3<AND2>(b[33], q21, 0u);
            const uint32_t m1 = lop3<AND2>(b[63], b[45], 0u);
            const uint32_t m2 = lop3<AND2>(b[28], b[9], 0u);
            const uint32_t a2 = lop3<XAND>(t3, m1, m2);
            const uint32_t p7 = lop3<AND3>(b[60], b[52], p2);
            const uint32_t p8 = lop3<AND3>(p1, b[21], b[15]);
            const uint32_t p9 = lop3<AND3>(p1, q45, b[37]);
            const uint32_t a3 = lop3<XAND>(t4, p5, p3);
            const uint32_t p11 = lop3<AND3>(q45, p2, q21);
            const uint32_t u1 = lop3<XOR3>(t1, a1, a2);
            const uint32_t u2 = lop3<XOR3>(a3, p1, p2);
            const uint32_t u3 = lop3<XOR3>(p3, p5, p7);
            const uint32_t u4 = lop3<XOR3>(p8, p9, p11);
            const uint32_t gb = lop3<XOR3>(lop3<XOR3>(u1, u2, u3), u4, 0u);
            // h + z (9 + 1)
            const uint32_t x0 = s3, x1 = s25, x2 = s46, x3 = s64, x4 = b[63];
            const uint32_t m = lop3<MUX>(x3, x0, x4);
            const uint32_t B0 = lop3<0xE4u>(x1, x3, x4);
            const uint32_t B1 = lop3<0x72u>(x1, x3, x4);
            const uint32_t B = lop3<MUX>(x0, B1, B0);
            const uint32_t w1 = lop3<XOR3>(b[1], b[2], b[4]);
            const uint32_t w2 = lop3<XOR3>(b[10], b[31], b[43]);
            const uint32_t w3 = lop3<XOR3>(b[56], x1, m);
            uint32_t w = lop3<XOR3>(w1, w2, w3);
            w = lop3<XOR2>(w, acc, 0u);
            acc = lop3<XAND>(w, x2, B);
            if (FULL) {
                const uint32_t fs = lop3<XOR3>(lop3<XOR3>(s[62], s[51], s[38]), lop3<XOR3>(s[23], s[13], s[0]), 0u);
#pragma unroll
                for (int i = 0; i < 79; ++i) s[i] = s[i + 1];
                s[79] = fs;
            }
#pragma unroll
            for (int i = 0; i < 79; ++i) b[i] = b[i + 1];
            b[79] = gb;
        }
        base += 32;
    }
    uint32_t r = acc;
#pragma unroll
    for (int i = 0; i < 80; ++i) r ^= b[i] ^ (FULL ? s[i] : 0u);
    out[blockIdx.x * 128 + tid] = r;
}

int main(int argc, char** argv)
{
    const double mhz = argc > 1 ? atof(argv[1]) : 1965.0;
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    uint32_t* out;
    cudaMalloc(&out, sms * 128 * 4);
    const int iters = 4096;  // x 32 clocks
    cudaFuncSetAttribute(probe<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 256 * 128 * 4);
    cudaFuncSetAttribute(probe<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 256 * 128 * 4);
    for (int full = 0; full < 2; ++full) {
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        float best = 1e30f;
        for (int r = 0; r < 4; ++r) {
            cudaEventRecord(a);
            if (full)
                probe<true><<<sms, 128, 256 * 128 * 4>>>(out, iters, 7 + r);
            else
                probe<false><<<sms, 128, 256 * 128 * 4>>>(out, iters, 7 + r);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            if (ms < best) best = ms;
        }
        const double clocks = double(iters) * 32;
        printf("{\"probe\": \"%s\", \"ms\": %.3f, \"cycles_per_clock\": %.1f}\n",
               full ? "whole Grain (lone warp)" : "NFSR half, LFSR taps from smem (lone warp)", best,
               best * 1e-3 * mhz * 1e6 / clocks);
    }
    return 0;
}
