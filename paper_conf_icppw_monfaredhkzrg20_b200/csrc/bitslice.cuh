// bitslice.cuh -- layout conversions for the column-major ("bitsliced")
// representation, sm_100a.
//
// PAPER.md:478-489 (sec. 4.1): "a batch of 32 bits data stored in a single
// register, represents state bits from 32 uncorrelated different parallel
// LFSRs having the same bit significance".  Lane j of a slice word is instance
// 32g + j of group g (reading R8).
#pragma once
#include <cstdint>

namespace bsk {

// One explicit 3-input logic op: d = LUT(a, b, c), LUT bit 4a+2b+c
// (truth tables written as F(0xF0, 0xCC, 0xAA)).  Inline PTX keeps the
// compiler from re-associating hand-chosen LOP3 trees.
template <uint32_t LUT>
__device__ __forceinline__ uint32_t lop3(uint32_t a, uint32_t b, uint32_t c)
{
    uint32_t d;
    asm("lop3.b32 %0, %1, %2, %3, %4;" : "=r"(d) : "r"(a), "r"(b), "r"(c), "n"(LUT));
    return d;
}

// ---------------------------------------------------------------------------
// Key/IV slicing (SURVEY step a-1; "32x80 bits of IV for each
// thread").  One warp per group g: lane j holds instance 32g+j's byte string;
// one __ballot_sync per bit position gathers the 32 lanes into a slice word.
//   raw   : uint8 [n][NBYTES] row-major (device)
//   out   : uint32 [NBITS][Gp]  (bit b of instance 32g+j -> bit j of out[b][g])
//   MSB   : bit b of a byte string is (byte[b/8] >> (7 - b%8)) & 1 if true
//           (MICKEY, spec [5]), (byte[b/8] >> (b%8)) & 1 otherwise (Grain)
// Instances >= n (padding) get all-zero bytes.
// ---------------------------------------------------------------------------
// Block = SLICE_GROUPS warps = that many consecutive groups; the ballot words
// are staged in shared memory as [bit][group] and written out as one 32 B DRAM
// sector per bit (per-warp 4-byte stores strided by Gp were 20x slower).  The
// first version used 1024-thread blocks (32 groups, one 128 B segment per
// bit): one resident block per SM left the loads' latency exposed (120 us per
// 2^22 keys); 256-thread blocks keep 8 blocks in flight per SM.
constexpr int SLICE_GROUPS = 8;
constexpr int SLICE_BLOCK = 32 * SLICE_GROUPS;

template <int NBYTES, int NBITS, bool MSB>
__global__ void __launch_bounds__(SLICE_BLOCK) slice_bits_kernel(const uint8_t* __restrict__ raw,
                                                                 uint64_t n, uint32_t* __restrict__ out,
                                                                 uint64_t Gp)
{
    __shared__ uint32_t tile[NBITS][SLICE_GROUPS];
    const uint32_t wib = threadIdx.x >> 5;
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t g0 = uint64_t(blockIdx.x) * SLICE_GROUPS;  // first group of this block
    const uint64_t warp = g0 + wib;
    if (warp < Gp) {  // warp-uniform
        const uint64_t inst = warp * 32u + lane;
        const uint8_t* src = raw + (inst < n ? inst : 0) * NBYTES;
        uint32_t b[NBYTES];
#pragma unroll
        for (int i = 0; i < NBYTES; ++i) b[i] = (inst < n) ? uint32_t(__ldg(src + i)) : 0u;
#pragma unroll
        for (int bit = 0; bit < NBITS; ++bit) {
            const uint32_t v = MSB ? (b[bit >> 3] >> (7 - (bit & 7))) & 1u : (b[bit >> 3] >> (bit & 7)) & 1u;
            const uint32_t w = __ballot_sync(0xffffffffu, v);
            if (lane == 0) tile[bit][wib] = w;
        }
    }
    __syncthreads();
    for (uint32_t idx = threadIdx.x; idx < uint32_t(NBITS) * SLICE_GROUPS; idx += SLICE_BLOCK) {
        const uint32_t bit = idx / SLICE_GROUPS, gw = idx % SLICE_GROUPS;
        if (g0 + gw < Gp) out[uint64_t(bit) * Gp + g0 + gw] = tile[bit][gw];
    }
}

// ---------------------------------------------------------------------------
// 32x32 bit transpose, one thread, in registers (SURVEY step a-4 (iii)).
// Input rows x[q] (q = 0..N-1) are a slab of the 32x32 matrix A after the
// stage-16 PRMT split; output x[q] = B[.] with B[c] bit r = A[r] bit c.
// Stages s = 8 (PRMT byte shuffle), 4, 2, 1 (shift + LOP3 select) on row pairs
// (r, r+s), r & s == 0.  16 rows -> 8 + 3*16 = 56... ops, all ALU.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void bt_stage8(uint32_t& a, uint32_t& b)
{
    const uint32_t na = __byte_perm(a, b, 0x6240);
    const uint32_t nb = __byte_perm(a, b, 0x7351);
    a = na;
    b = nb;
}

// b << S and a >> S as integer multiplies (IMAD / IMAD.HI on the FMA pipe):
// the keystream loop saturates the ALU pipe, the FMA pipe is idle.
template <int S>
__device__ __forceinline__ uint32_t shl_fma(uint32_t x)
{
    uint32_t d;
    asm("mul.lo.u32 %0, %1, %2;" : "=r"(d) : "r"(x), "n"(1u << S));
    return d;
}
template <int S>
__device__ __forceinline__ uint32_t shr_fma(uint32_t x)
{
    uint32_t d;
    asm("mul.hi.u32 %0, %1, %2;" : "=r"(d) : "r"(x), "n"(1u << (32 - S)));
    return d;
}

// d = M ? x : y bitwise, one LOP3 with M as its immediate operand.  Written
// as C `(x & M) | (y & ~M)` ptxas emits two LOP3s (an AND with the immediate,
// then an OR-AND with ~M): 96 extra ALU ops per 32x32 transpose.
template <uint32_t M>
__device__ __forceinline__ uint32_t sel_imm(uint32_t x, uint32_t y)
{
    uint32_t d;
    asm("lop3.b32 %0, %1, %2, %3, 0xE4;" : "=r"(d) : "r"(x), "r"(y), "n"(M));  // c ? a : b
    return d;
}

// d = m ? x : y bitwise, m in a register: one LOP3 (0xCA: a ? b : c)
__device__ __forceinline__ uint32_t sel_imm_var(uint32_t m, uint32_t x, uint32_t y)
{
    uint32_t d;
    asm("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(d) : "r"(m), "r"(x), "r"(y));
    return d;
}

template <int S, uint32_t M>
__device__ __forceinline__ void bt_stage(uint32_t& a, uint32_t& b)
{
    // element (r, c | S) <-> (r + S, c), c & S == 0; M = bits with c & S == 0
    const uint32_t na = sel_imm<M>(a, shl_fma<S>(b));
    const uint32_t nb = sel_imm<M>(shr_fma<S>(a), b);
    a = na;
    b = nb;
}

// Transpose the 16-row half produced by the stage-16 split.
__device__ __forceinline__ void bt_transpose16(uint32_t (&x)[16])
{
#pragma unroll
    for (int r = 0; r < 16; ++r)
        if ((r & 8) == 0) bt_stage8(x[r], x[r + 8]);
#pragma unroll
    for (int r = 0; r < 16; ++r)
        if ((r & 4) == 0) bt_stage<4, 0x0F0F0F0Fu>(x[r], x[r + 4]);
#pragma unroll
    for (int r = 0; r < 16; ++r)
        if ((r & 2) == 0) bt_stage<2, 0x33333333u>(x[r], x[r + 2]);
#pragma unroll
    for (int r = 0; r < 16; ++r)
        if ((r & 1) == 0) bt_stage<1, 0x55555555u>(x[r], x[r + 1]);
}

// ---------------------------------------------------------------------------
// Per-thread key/IV slicing for fused init kernels (SURVEY step a-1 inside
// a-2).  Thread = one group of 32 instances, as in the clock loop.  `p` =
// the group's 32 byte strings (32*NBYTES bytes, 16 B aligned, zero-padded past
// n).  For each 32-bit chunk c the thread builds A[j] = bytes 4c..4c+3 of
// instance j (big-endian if MSB, so string bit 32c+t is A bit 31-t; else
// little-endian, bit 32c+t = A bit t), transposes the 32x32 block in
// registers (bt_transpose16: B[r] bit j = A[j] bit r) and hands every slice
// word to put(bit, word): bit 32c+31-r (MSB) or 32c+r (LSB).  The group's
// bytes are read with 16 B loads straight into registers (no smem staging).
// ---------------------------------------------------------------------------
// Where group g's 32 byte strings live: groups g < g_split straight in the
// caller's row-major input (device inputs, no staging copy), the rest (the
// partial last group and the padding groups) in a zero-padded tail buffer.
__device__ __forceinline__ const uint8_t* group_src(const uint8_t* main, const uint8_t* tail, uint64_t g_split,
                                                    uint64_t g, uint32_t group_bytes)
{
    return g < g_split ? main + g * group_bytes : tail + (g - g_split) * group_bytes;
}

// Stage a warp's 32 consecutive group blocks (GB bytes each, contiguous in
// global memory from `src`) into shared memory, one row of STRIDE bytes per
// lane, with coalesced 16 B loads (512 contiguous bytes per instruction).
// Per-thread 16 B loads of the own 320 B block touch 32 lines per instruction
// (8x the L1 wavefronts); ncu: long-scoreboard stalls at 0.31 per issue in
// the Grain init kernel.  STRIDE = GB + 16 keeps the lanes' 16 B smem reads
// of their own rows bank-conflict free.
template <int GB, int STRIDE>
__device__ __forceinline__ void stage_warp_groups(const uint8_t* __restrict__ src, uint8_t* dst, uint32_t lane)
{
    static_assert(GB % 16 == 0 && STRIDE % 16 == 0, "16 B pieces");
    constexpr int PIECES = GB / 16;
    const uint4* s = reinterpret_cast<const uint4*>(src);
#pragma unroll
    for (int k = 0; k < PIECES; ++k) {
        const uint32_t P = lane + 32u * k;
        const uint4 v = __ldcs(s + P);
        *reinterpret_cast<uint4*>(dst + (P / PIECES) * STRIDE + (P % PIECES) * 16) = v;
    }
}
// The same for one lane's own block (warps whose groups are not contiguous).
template <int GB, int STRIDE>
__device__ __forceinline__ void stage_own_group(const uint8_t* __restrict__ src, uint8_t* dst, uint32_t lane)
{
    const uint4* s = reinterpret_cast<const uint4*>(src);
#pragma unroll
    for (int k = 0; k < GB / 16; ++k) *reinterpret_cast<uint4*>(dst + lane * STRIDE + 16 * k) = __ldcs(s + k);
}

// GLOBAL: p is global memory (streaming 16 B loads); else shared memory.
template <int NBYTES, int NBITS, bool MSB, bool GLOBAL = true, class Put>
__device__ __forceinline__ void slice_group32(const uint8_t* __restrict__ p, Put&& put)
{
    static_assert((32 * NBYTES) % 16 == 0, "group block must be whole 16 B vectors");
    constexpr int NW = 32 * NBYTES / 4;
    uint32_t raw[NW + 1];
    const uint4* src = reinterpret_cast<const uint4*>(p);
#pragma unroll
    for (int i = 0; i < NW / 4; ++i) {
        const uint4 v = GLOBAL ? __ldcs(src + i) : src[i];
        raw[4 * i] = v.x;
        raw[4 * i + 1] = v.y;
        raw[4 * i + 2] = v.z;
        raw[4 * i + 3] = v.w;
    }
    raw[NW] = 0u;  // straddle guard for the last instance's final chunk
    constexpr int NCHUNK = (NBITS + 31) / 32;
#pragma unroll
    for (int c = 0; c < NCHUNK; ++c) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            // rows r = 16h + q; skip halves whose bits are all >= NBITS
            const int lo_bit = MSB ? 32 * c + 31 - (16 * h + 15) : 32 * c + 16 * h;
            if (lo_bit >= NBITS) continue;
            uint32_t x[16];
#pragma unroll
            for (int q = 0; q < 16; ++q) {
                uint32_t a2[2];
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    const int j = q + 16 * e;
                    const int bo = NBYTES * j + 4 * c;
                    const int w0 = bo / 4, off = bo % 4;
                    const uint32_t sel = MSB ? ((uint32_t(off) << 12) | (uint32_t(off + 1) << 8) |
                                                (uint32_t(off + 2) << 4) | uint32_t(off + 3))
                                             : ((uint32_t(off + 3) << 12) | (uint32_t(off + 2) << 8) |
                                                (uint32_t(off + 1) << 4) | uint32_t(off));
                    a2[e] = __byte_perm(raw[w0], off ? raw[w0 + 1] : 0u, sel);
                }
                x[q] = __byte_perm(a2[0], a2[1], h == 0 ? 0x5410 : 0x7632);
            }
            bt_transpose16(x);  // x[q] = B[16h + q]
#pragma unroll
            for (int q = 0; q < 16; ++q) {
                const int bit = MSB ? 32 * c + 31 - (16 * h + q) : 32 * c + 16 * h + q;
                if (bit < NBITS) put(bit, x[q]);
            }
        }
    }
}

// Slice 32-instance group blocks straight into state rows [bit][Gp] (AES-CTR
// initial counters, LFSR keys: the sliced input IS the state).  One thread
// per group; raw = Gp*32 rows of NBYTES, 16 B aligned, zero past n.
// The warp's group blocks are staged through shared memory with coalesced
// loads (stage_warp_groups); SS_SMEM_BYTES(NBYTES) of dynamic smem per CTA.
__host__ __device__ constexpr int ss_stride(int nbytes) { return 32 * nbytes + 16; }
__host__ __device__ constexpr size_t ss_smem_bytes(int nbytes) { return size_t(128) * ss_stride(nbytes); }

template <int NBYTES, int NBITS, bool MSB>
__global__ void __launch_bounds__(128) slice_state_kernel(const uint8_t* __restrict__ raw,
                                                          const uint8_t* __restrict__ tail, uint64_t g_split,
                                                          uint32_t* __restrict__ state, uint64_t Gp)
{
    constexpr int GB = 32 * NBYTES, STRIDE = ss_stride(NBYTES);
    extern __shared__ __align__(16) uint8_t ss_smem[];
    const uint64_t g = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
    if (g >= Gp) return;  // whole warps (Gp is a multiple of 32)
    const uint32_t lane = threadIdx.x & 31u;
    uint8_t* w = ss_smem + (threadIdx.x >> 5) * 32 * STRIDE;
    const uint64_t g0 = g - lane;
    if (g0 + 32 <= g_split)
        stage_warp_groups<GB, STRIDE>(raw + g0 * GB, w, lane);
    else
        stage_own_group<GB, STRIDE>(group_src(raw, tail, g_split, g, GB), w, lane);
    __syncwarp();
    uint32_t* p = state + g;
    slice_group32<NBYTES, NBITS, MSB, false>(w + lane * STRIDE, [&](int bit, uint32_t v) { p[uint64_t(bit) * Gp] = v; });
}

// Hide a pointer's provenance from the optimiser (no code emitted beyond a
// register move), so address arithmetic is not hoisted/CSE'd across the
// register-resident clock loop.
template <class T>
__device__ __forceinline__ T* opaque(T* p)
{
    asm volatile("" : "+l"(p));
    return p;
}

__device__ __forceinline__ uint64_t fmix64(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

}  // namespace bsk
