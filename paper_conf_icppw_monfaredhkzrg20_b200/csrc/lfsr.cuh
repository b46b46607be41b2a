// lfsr.cuh -- the paper's bitsliced LFSR, sm_100a.
//
// PAPER.md:578-596 (sec. 4.3, Fig. 8): "the bitsliced LFSR implementation with
// column-major representation ... executed by a single thread ... the 32 x k
// number of costly bit-wise XOR operations is reduced to k number of full-width
// XOR operations ... the costly bit-level shift operations are replaced by ...
// register swapping".  Polynomial (reading L1): p(x) = x^128 + x^29 + x^27 +
// x^2 + 1, primitive; Fibonacci form s_{t+128} = s_{t+29} ^ s_{t+27} ^ s_{t+2}
// ^ s_t, output z_t = s_t.  Per clock: 2 LOP3 for 32 keystream bits (k = 4
// taps); the shift is renaming, closed by 128/U moves per clock (FMA pipe).
// With so little logic the materialised keystream is bound by HBM writes --
// this workload exercises the output path at the memory roofline.
#pragma once
#include <cstdint>

#include "bitslice.cuh"

namespace bsk {

struct Lfsr128 {
    static constexpr int NSTATE = 128;
    static constexpr bool MSB_FIRST = true;
    static constexpr int U_DEFAULT = 32, U_ALT0 = 16, U_ALT1 = 16;
    static constexpr bool RM_TMEM = false, RM_SEGMENTED = true;
    // ROW_MAJOR: always a warp-specialised kernel (2 LOP3 per clock leave the
    // output path as the whole cost): two writer warps per clock-loop warp,
    // two streams per SM, 128 B row pieces written as sector pairs
    // (rowmajor_ws2.cuh; C2 27.5 Tb/s), rather than one writer per stream with
    // 64 B pieces (rowmajor_ws.cuh, 26.3; 11.9 with 32 B smem staging)
    static constexpr int RM_WS = 3;
    // consume: one 128-clock body (the rotation period), no moves (keystream.cuh)
    static constexpr int U_CONSUME = 128;
    static constexpr bool CONSUME_PERIOD = true;
    uint32_t s[128];

    __device__ __forceinline__ void load(const uint32_t* st, uint64_t Gp, uint64_t g)
    {
        const uint32_t* p = opaque(st + g);
#pragma unroll
        for (int i = 0; i < 128; ++i) s[i] = __ldcg(p + uint64_t(i) * Gp);
    }
    __device__ __forceinline__ void store(uint32_t* st, uint64_t Gp, uint64_t g) const
    {
        uint32_t* p = opaque(st + g);
#pragma unroll
        for (int i = 0; i < 128; ++i) __stcg(p + uint64_t(i) * Gp, s[i]);
    }
    __device__ __forceinline__ uint32_t z() const { return s[0]; }
    __device__ __forceinline__ uint32_t z_acc(uint32_t acc) const { return acc ^ s[0]; }
    // One consume period: 128 clocks with their output words XORed into acc.
    // The outputs of clocks t = 0..127 are z_t = s_t, i.e. exactly the 128
    // state words at entry, so they are folded first (43 XOR3 in a 3-ary
    // tree) and the 128 clocks then run in place: register t takes s_{t+128}
    // = s_t ^ s_{t+2} ^ s_{t+27} ^ s_{t+29}, whose operands sit in registers
    // (t+k) mod 128 (already overwritten iff t+k >= 128, which is then the
    // needed s_{t+k}).  Same 2.5 ops per clock as the per-clock form, but no
    // register outlives its clock, so no moves.
    __device__ __forceinline__ void consume_period(uint32_t& acc)
    {
        uint32_t r[43];
#pragma unroll
        for (int i = 0; i < 42; ++i) r[i] = lop3<0x96u>(s[3 * i], s[3 * i + 1], s[3 * i + 2]);
        r[42] = lop3<0x96u>(s[126], s[127], acc);
        uint32_t q[15];
#pragma unroll
        for (int i = 0; i < 14; ++i) q[i] = lop3<0x96u>(r[3 * i], r[3 * i + 1], r[3 * i + 2]);
        q[14] = r[42];
        uint32_t p[5];
#pragma unroll
        for (int i = 0; i < 5; ++i) p[i] = lop3<0x96u>(q[3 * i], q[3 * i + 1], q[3 * i + 2]);
        acc = lop3<0x96u>(lop3<0x96u>(p[0], p[1], p[2]), p[3], p[4]);
#pragma unroll
        for (int t = 0; t < 128; ++t)
            s[t] = lop3<0x96u>(lop3<0x96u>(s[(t + 29) & 127], s[(t + 27) & 127], s[(t + 2) & 127]), s[t], 0u);
    }
    // ROW_MAJOR period body (rowmajor_ws.cuh), block J = clocks 32J..32J+31
    // of a 128-clock period: their outputs are the entry state words
    // s[32J..32J+31] (handed to put(u, word)), after which those registers are
    // clocked in place as in consume_period (registers of later blocks still
    // hold their entry words when their block comes).  No moves.
    static constexpr int PERIOD_BLOCKS = 4;
    template <int J, class F>
    __device__ __forceinline__ void period_block(F&& put)
    {
        // u as a compile-time constant (the writer-warp kernels group 4 per STS.128)
        static_for<32>([&](auto u) { put(u, s[32 * J + decltype(u)::value]); });
#pragma unroll
        for (int t = 32 * J; t < 32 * J + 32; ++t)
            s[t] = lop3<0x96u>(lop3<0x96u>(s[(t + 29) & 127], s[(t + 27) & 127], s[(t + 2) & 127]), s[t], 0u);
    }
    __device__ __forceinline__ void clock()
    {
        const uint32_t fb = lop3<0x96u>(lop3<0x96u>(s[29], s[27], s[2]), s[0], 0u);
#pragma unroll
        for (int i = 0; i < 127; ++i) s[i] = s[i + 1];
        s[127] = fb;
    }
};

}  // namespace bsk
