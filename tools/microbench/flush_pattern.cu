// flush_pattern.cu -- HBM write rate of the ROW_MAJOR flush patterns, without
// any keystream compute (which store shape can the materialise kernels use?).
//
// The keystream kernels' output: warp w owns 32 groups = 1024 instance rows
// (rows 1024 w .. 1024 w + 1023, pitch P bytes) and every 256 clocks writes one
// 32 B sector (column c) of each of its 1024 rows.  Persistent grid, WARPS
// resident warps per SM, each walking its rows' columns.  Variants (one store
// instruction always writes whole 32 B sectors):
//   quad_g : STG.64, 4 lanes per row, the 8 rows of an instruction are 8
//            groups apart (the tcgen05.ld.16x256b read-back: rowmajor_store_tmem_sectors)
//   quad_q : STG.64, 4 lanes per row, 8 consecutive rows (same group)
//   pair_g : STG.128, 2 lanes per row, 16 rows 1 group apart each
//   pair_q : STG.128, 2 lanes per row, 16 consecutive rows
//   one    : STG.128 x2, 1 lane per row (half sectors per instruction)
// Prints one JSON line per variant: best of 5, CUDA events.
#include <cstdint>
#include <cstdio>

enum { QUAD_G, QUAD_Q, PAIR_G, PAIR_Q, ONE, SEG64, SEG128, SEG256, MIX, SPLIT128, SEG64_2W };
// SPLIT128: warps 2p, 2p+1 of a CTA share one unit of 1024 rows; every flush
//   writes 128 B of each row, warp 2p the row's 32 B sectors 0 and 2, warp
//   2p+1 sectors 1 and 3 (16x256b-style: 4 lanes x 16 B per row, 8 rows per
//   STG.128) -- two writer warps in two TMEM lane quarters per stream
// SEG64_2W: SEG64 with only 2 of the 4 warps of a CTA working (half the rows
//   in flight per SM)
// store cache policy: 0 = evict-first (st.global.cs), 1 = default (write-back,
// L2 evict_normal), 2 = L2 evict_last (createpolicy)
template <int POL>
__device__ __forceinline__ void st64(void* p, uint2 v)
{
    if constexpr (POL == 0) {
        __stcs(reinterpret_cast<uint2*>(p), v);
    } else if constexpr (POL == 1) {
        *reinterpret_cast<uint2*>(p) = v;
    } else {
        uint64_t pol;
        asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
        asm volatile("st.global.L2::cache_hint.v2.u32 [%0], {%1, %2}, %3;" ::"l"(p), "r"(v.x), "r"(v.y), "l"(pol)
                     : "memory");
    }
}
template <int POL>
__device__ __forceinline__ void st128(void* p, uint4 v)
{
    if constexpr (POL == 0) {
        __stcs(reinterpret_cast<uint4*>(p), v);
    } else if constexpr (POL == 1) {
        *reinterpret_cast<uint4*>(p) = v;
    } else {
        uint64_t pol;
        asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
        asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p), "r"(v.x), "r"(v.y),
                     "r"(v.z), "r"(v.w), "l"(pol)
                     : "memory");
    }
}

template <int V, int POL>
__global__ void __launch_bounds__(128) flush_kernel(uint8_t* out, uint64_t pitch, uint32_t units, uint32_t seed)
{
    const uint32_t lane = threadIdx.x & 31;
    if (V == SPLIT128 || V == SEG64_2W) {
        const uint32_t wi = threadIdx.x >> 5;
        if (V == SEG64_2W && (wi & 1)) return;
        const uint32_t npairs = gridDim.x * 2;
        const uint32_t half = wi & 1;
        for (uint32_t w = blockIdx.x * 2 + (wi >> 1); w < units; w += npairs) {
            uint8_t* base = out + uint64_t(w) * 1024 * pitch;
            const uint32_t bpr = V == SPLIT128 ? 128 : 64;
            for (uint64_t c = 0; c < pitch; c += bpr) {
                const uint32_t v = seed ^ uint32_t(c) ^ w;
#pragma unroll 4
                for (uint32_t it = 0; it < 128; ++it) {
                    const uint32_t row = it * 8 + (lane >> 2), j = lane & 3;
                    const uint32_t off = V == SPLIT128 ? 32 * (2 * (j >> 1) + half) + 16 * (j & 1) : 16 * j;
                    st128<POL>(base + uint64_t(row) * pitch + c + off, make_uint4(v, it, lane, 5));
                }
            }
        }
        return;
    }
    const uint32_t nwarps = gridDim.x * 4;
    for (uint32_t w = blockIdx.x * 4 + (threadIdx.x >> 5); w < units; w += nwarps) {
        uint8_t* base = out + uint64_t(w) * 1024 * pitch;
        for (uint64_t c = 0; c < pitch; c += 32) {
            const uint32_t v = seed ^ uint32_t(c) ^ w;
            if (V == QUAD_G) {
                // rows (group 8i + lane/4 (+ 16 * h), q): instruction = 8 groups at one q
#pragma unroll 4
                for (uint32_t it = 0; it < 128; ++it) {
                    const uint32_t q = it & 31, gb = (it >> 5) * 8;
                    uint8_t* p = base + uint64_t(32 * (gb + (lane >> 2)) + q) * pitch + c + 8 * (lane & 3);
                    st64<POL>(p, make_uint2(v, it));
                }
            } else if (V == QUAD_Q) {
#pragma unroll 4
                for (uint32_t it = 0; it < 128; ++it) {
                    const uint32_t row = it * 8 + (lane >> 2);
                    uint8_t* p = base + uint64_t(row) * pitch + c + 8 * (lane & 3);
                    st64<POL>(p, make_uint2(v, it));
                }
            } else if (V == PAIR_G) {
#pragma unroll 4
                for (uint32_t it = 0; it < 64; ++it) {
                    const uint32_t q = it & 31, gb = (it >> 5) * 16;
                    uint8_t* p = base + uint64_t(32 * (gb + (lane >> 1)) + q) * pitch + c + 16 * (lane & 1);
                    st128<POL>(p, make_uint4(v, it, lane, 1));
                }
            } else if (V == PAIR_Q) {
#pragma unroll 4
                for (uint32_t it = 0; it < 64; ++it) {
                    const uint32_t row = it * 16 + (lane >> 1);
                    uint8_t* p = base + uint64_t(row) * pitch + c + 16 * (lane & 1);
                    st128<POL>(p, make_uint4(v, it, lane, 1));
                }
            } else if (V == MIX) {
                // warps 0-3 of each 8-warp SM: 64 B per row per flush (4 lanes x
                // 16 B, 8 rows per STG.128); warps 4-7: 32 B (4 lanes x 8 B)
                const bool wide = (blockIdx.x & 1) == 0;  // 2 CTAs per SM: one wide, one narrow
                if (wide) {
                    if (c % 64) continue;
#pragma unroll 4
                    for (uint32_t it = 0; it < 128; ++it) {
                        const uint32_t row = it * 8 + (lane >> 2);
                        st128<POL>(base + uint64_t(row) * pitch + c + 16 * (lane & 3), make_uint4(v, it, lane, 3));
                    }
                } else {
#pragma unroll 4
                    for (uint32_t it = 0; it < 128; ++it) {
                        const uint32_t row = it * 8 + (lane >> 2);
                        st64<POL>(base + uint64_t(row) * pitch + c + 8 * (lane & 3), make_uint2(v, it));
                    }
                }
            } else if (V >= SEG64) {
                // BPR bytes per row per flush (c advances by BPR), 16 B per lane:
                // one instruction = 512 / BPR consecutive rows x BPR contiguous bytes
                constexpr uint32_t BPR = V == SEG64 ? 64 : V == SEG128 ? 128 : 256, LPR = BPR / 16;
                if (c % BPR) continue;
#pragma unroll 4
                for (uint32_t it = 0; it < 1024 / (32 / LPR); ++it) {
                    const uint32_t row = it * (32 / LPR) + lane / LPR;
                    uint8_t* p = base + uint64_t(row) * pitch + c + 16 * (lane % LPR);
                    st128<POL>(p, make_uint4(v, it, lane, 2));
                }
            } else {
#pragma unroll 4
                for (uint32_t q = 0; q < 32; ++q) {
                    uint8_t* p = base + uint64_t(32 * lane + q) * pitch + c;
                    st128<POL>(p, make_uint4(v, q, lane, 0));
                    st128<POL>(reinterpret_cast<uint4*>(p) + 1, make_uint4(v, q, lane, 1));
                }
            }
        }
    }
}

template <int V, int POL>
void run(const char* name, uint8_t* buf, uint64_t pitch, uint32_t units, int sms, int ctas)
{
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int r = 0; r < 6; ++r) {
        cudaEventRecord(a);
        flush_kernel<V, POL><<<sms * ctas, 128>>>(buf, pitch, units, 0x9E3779B9u + r);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (r > 0 && ms < best) best = ms;
    }
    const double bytes = double(units) * 1024 * pitch;
    printf("{\"pattern\": \"%s\", \"policy\": \"%s\", \"pitch\": %llu, \"warps_per_sm\": %d, \"bytes\": %.0f, \"ms\": %.3f, \"write_gbs\": %.1f}\n",
           name, POL == 0 ? "evict_first" : POL == 1 ? "default" : "evict_last", (unsigned long long)pitch, 4 * ctas, bytes, best, bytes / (best * 1e-3) / 1e9);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
}

int main()
{
    const uint64_t nbytes = uint64_t(16) << 30;
    uint8_t* buf;
    if (cudaMalloc(&buf, nbytes) != cudaSuccess) { printf("{\"error\": \"cudaMalloc\"}\n"); return 1; }
    int sms = 148;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (uint64_t pitch : {uint64_t(4096), uint64_t(32768)}) {
        const uint32_t units = uint32_t(nbytes / (1024 * pitch));
        for (int ctas : {1, 2}) {
            if (ctas == 2 && pitch > 4096) continue;
            run<QUAD_G, 0>("quad_g", buf, pitch, units, sms, ctas);
            run<QUAD_G, 1>("quad_g", buf, pitch, units, sms, ctas);
            run<QUAD_G, 2>("quad_g", buf, pitch, units, sms, ctas);
            run<PAIR_Q, 0>("pair_q", buf, pitch, units, sms, ctas);
            run<PAIR_Q, 1>("pair_q", buf, pitch, units, sms, ctas);
            run<PAIR_Q, 2>("pair_q", buf, pitch, units, sms, ctas);
            run<ONE, 1>("one", buf, pitch, units, sms, ctas);
            run<SEG64, 0>("seg64", buf, pitch, units, sms, ctas);
            run<SEG64, 2>("seg64", buf, pitch, units, sms, ctas);
            run<SEG128, 0>("seg128", buf, pitch, units, sms, ctas);
            run<SEG128, 2>("seg128", buf, pitch, units, sms, ctas);
            run<SEG256, 0>("seg256", buf, pitch, units, sms, ctas);
            if (ctas == 1) {
                run<SPLIT128, 2>("split128_2streams", buf, pitch, units, sms, ctas);
                run<SPLIT128, 1>("split128_2streams", buf, pitch, units, sms, ctas);
                run<SEG64_2W, 2>("seg64_2streams", buf, pitch, units, sms, ctas);
            }
            if (ctas == 2) {
                run<MIX, 0>("mix_64_32", buf, pitch, units, sms, ctas);
                run<MIX, 2>("mix_64_32", buf, pitch, units, sms, ctas);
            }
        }
    }
    cudaFree(buf);
    return 0;
}
