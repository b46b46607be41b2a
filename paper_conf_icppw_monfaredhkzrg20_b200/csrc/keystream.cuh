// keystream.cuh -- the register-resident keystream clock loop (SURVEY steps a-3,
// a-4, a-5), generic over a bitsliced cipher C, for sm_100a.
//
// One thread = one group of 32 instances = one slice word per state bit
// (PAPER.md:618-626).  The whole state lives in registers across all clocks of
// a work item ("do not require any additional memory rather
// than registers"); it touches HBM only at item entry/exit (state carry, a-5).
//
// Work distribution (B200 design, not the paper's): a persistent grid sized to
// the resident-warp capacity of the 148 SMs pulls work items from an atomic
// ticket.  Item k = (segment k / units, warp-unit k % units): 32 groups for
// seg_clocks clocks.  Segment s of a unit waits for segment s-1 of the same
// unit (flag), so a call is split in time as well as across instances and the
// last wave's tail is one segment long instead of one whole call.  Tickets are
// taken in order by resident warps, so every awaited item is held by a running
// warp: no deadlock.
//
// Output layouts (sec. 4.5: registers -> shared memory ->
// coalesced global stores):
//   CHECKSUM : acc ^= z (fused into the output LOP3); fmix64 + warp sum + one
//              atomicAdd per warp at the end of the call.
//   SLICED   : out[t][g] = z -- one coalesced STG.32 per clock (128 B per warp).
//   ROW_MAJOR: z -> shared memory (one conflict-free STS per clock); every 32
//              clocks each thread reloads its 32 words, transposes the 32x32
//              bit block in registers (PRMT + shift/LOP3 butterfly, split in
//              two 16-row halves to bound register pressure) and writes one
//              32-bit word per instance row.
#pragma once
#include <cuda.h>  // CUtensorMap (type only; encoded on the host via the runtime's driver entry point)

#include <cstdint>
#include <type_traits>
#include <utility>

#include "bitslice.cuh"

namespace bsk {

// Per-clock calls of a U-clock loop body.  A cipher with a multi-clock
// schedule (MICKEY 2.0's deferred R reduction, mickey2.cuh) declares
// block_k(U) and clocks J = 0..K-1 of each K-clock block are compile-time
// phases (z_at / z_acc_at / clock_at); any other cipher uses z / z_acc / clock.
template <class C, class = void>
struct ks_phased : std::false_type {};
template <class C>
struct ks_phased<C, std::void_t<decltype(C::block_k(1))>> : std::true_type {};
template <class C, int U>
__host__ __device__ constexpr int ks_block()
{
    if constexpr (ks_phased<C>::value)
        return C::block_k(U);
    else
        return 1;
}
// Consume-mode clocks per iteration for ciphers whose register rotation
// closes after a short period (Lfsr128: 128 clocks, 3 LOP3 per clock): a body
// of the full period needs no rotation moves, which at U = 32 outnumber the
// logic (4 moves per clock).  0 = use U.
template <class C, class = void>
struct ks_u_big : std::integral_constant<int, 0> {};
template <class C>
struct ks_u_big<C, std::void_t<decltype(C::U_CONSUME)>> : std::integral_constant<int, C::U_CONSUME> {};
// A cipher whose consume body is a whole period may supply consume_period(acc)
// (Lfsr128: outputs folded from the entry state, clocks in place).
template <class C, class = void>
struct ks_period : std::false_type {};
template <class C>
struct ks_period<C, std::void_t<decltype(C::CONSUME_PERIOD)>> : std::integral_constant<bool, C::CONSUME_PERIOD> {};

template <int J, int K, class C>
__device__ __forceinline__ uint32_t ks_z(const C& c)
{
    if constexpr (K > 1)
        return c.template z_at<J, K>();
    else
        return c.z();
}
template <int J, int K, class C>
__device__ __forceinline__ uint32_t ks_z_acc(const C& c, uint32_t acc)
{
    if constexpr (K > 1)
        return c.template z_acc_at<J, K>(acc);
    else
        return c.z_acc(acc);
}
template <int J, int K, class C>
__device__ __forceinline__ void ks_clock(C& c)
{
    if constexpr (K > 1)
        c.template clock_at<J, K>();
    else
        c.clock();
}
template <class F, int... I>
__device__ __forceinline__ void static_for_impl(F&& f, std::integer_sequence<int, I...>)
{
    (f(std::integral_constant<int, I>{}), ...);
}
// f(integral_constant<int, i>) for i = 0..N-1, fully unrolled
template <int N, class F>
__device__ __forceinline__ void static_for(F&& f)
{
    static_for_impl(f, std::make_integer_sequence<int, N>{});
}

enum : int { L_ROW_MAJOR = 0, L_SLICED = 1, L_CHECKSUM = 2 };

struct KsArgs {
    uint32_t* state;      // [C::NSTATE + 1][Gp] (last row: checksum accumulator)
    uint64_t Gp;          // padded groups (multiple of 32) = 32 * units
    uint64_t G;           // real groups
    uint64_t n;           // real instances
    uint32_t tail_mask;   // valid lanes of group G-1
    uint64_t nclocks;     // clocks in this call (multiple of 32)
    uint64_t t0;          // clocks generated before this call
    uint64_t g_base;      // global index of group 0 (checksum)
    void* out;
    uint64_t row_bytes;   // ROW_MAJOR row stride = nclocks / 8
    uint64_t seg_clocks;  // clocks per work item (multiple of 32)
    uint64_t nseg;        // segments per call
    uint64_t units;       // warp-units = Gp / 32
    uint32_t* ticket;     // persistent mode: [1], zeroed before launch
    uint32_t* flags;      // persistent mode: [units], zeroed before launch
    uint32_t* scratch;    // [32] sink for padding-group SLICED stores
    unsigned long long* dbg;  // optional scheduler counters (BSRNG_DEBUG), or null
    int persistent;
    // ROW_MAJOR + TMEM: whole-sector flushes of warps whose 32 groups are all
    // real (g < tma_groups) go out as TMA tensor stores (rowmajor_store_tmem_tma)
    int use_tma;
    // ROW_MAJOR + TMEM with one CTA per SM (grid <= SMs, no time segments):
    // 512 columns = two staging buffers; a completed sector period is
    // flushed 4 rows per block during the next period (lone clock-loop warps
    // cannot otherwise hide the flush)
    int tmem_dbl;
    // ROW_MAJOR 32 B flushes (TMA / 8 B sector stores): L2 evict_last hint
    int l2last;
    // writer-warp kernel: stagger the units' 64 B flush periods (rowmajor_ws.cuh
    // ws::phase) so that they do not all flush in the same block
    int rm_phase;
    uint64_t tma_groups;
    CUtensorMap tmap;  // 3-D view of `out`: [q 32][group][byte], see bsrng.cu
};

__device__ __forceinline__ uint32_t ld_acquire(const uint32_t* p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release(uint32_t* p, uint32_t v)
{
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ uint32_t lane_mask(const KsArgs& a, uint64_t g)
{
    return g + 1 < a.G ? 0xFFFFFFFFu : (g + 1 == a.G ? a.tail_mask : 0u);
}

// ROW_MAJOR staging per warp (dynamic shared memory):
//   zs: z words of the current 32-clock block, [t][lane]      (4 KB / warp;
//       not used when the cipher loop keeps the block in registers, U = 32)
//   os: transposed words for one row segment of every row,
//       [row q][slot k][lane], k = 32-clock block within the segment
//       (SLOTS x 4 KB: SLOTS = 8 -> one whole 32 B DRAM sector per row,
//       SLOTS = 4 -> half a sector, half the smem, so two CTAs fit per SM)
// Every access is lane-contiguous, so STS/LDS are bank-conflict free.  Rows are
// written as whole 16 B pieces: 4-byte stores spread over the ~600k rows in
// flight overflowed L2 before their sectors filled, and the partial-sector
// evictions cost ~15x the algorithmic DRAM traffic (ncu).
constexpr int ZS_WORDS = 32 * 32;
constexpr int OS_WORDS = 32 * 8 * 32;  // SLOTS = 8
constexpr int RM_WARP_WORDS = ZS_WORDS + OS_WORDS;
__host__ __device__ constexpr int os_words(int slots) { return 32 * slots * 32; }
// zreg: the loop keeps its 32-clock z block in registers (U = 32 only)
__host__ __device__ constexpr int rm_warp_words(int U, int slots, bool zreg)
{
    return (U == 32 && zreg ? 0 : ZS_WORDS) + os_words(slots);
}

// Transpose this thread's 32 staged z words (a 32x32 bit block) and park the
// 32 row words in sector slot `k`.  Bit-matrix row t is clock t, or clock t^7
// for MSB-first ciphers so that clock 8b+q lands in bit 7-q of byte b.
template <bool MSB_FIRST, int SLOTS = 8>
__device__ __forceinline__ void rowmajor_transpose(const uint32_t* zs, uint32_t* os, uint32_t k)
{
    constexpr int X = MSB_FIRST ? 7 : 0;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t x[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) {
            const uint32_t lo = zs[(q ^ X) * 32];
            const uint32_t hi = zs[((q + 16) ^ X) * 32];
            x[q] = __byte_perm(lo, hi, h == 0 ? 0x5410 : 0x7632);
        }
        bt_transpose16(x);
#pragma unroll
        for (int q = 0; q < 16; ++q) os[((16 * h + q) * SLOTS + k) * 32] = x[q];
    }
}

// The same from 32 z words held in registers (cipher loops unrolled 32x).
template <bool MSB_FIRST, int SLOTS = 8>
__device__ __forceinline__ void rowmajor_transpose_regs(const uint32_t (&z)[32], uint32_t* os, uint32_t k)
{
    constexpr int X = MSB_FIRST ? 7 : 0;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t x[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) x[q] = __byte_perm(z[q ^ X], z[(q + 16) ^ X], h == 0 ? 0x5410 : 0x7632);
        bt_transpose16(x);
#pragma unroll
        for (int q = 0; q < 16; ++q) os[((16 * h + q) * SLOTS + k) * 32] = x[q];
    }
}

// 16 B row store: whole-sector flushes (SLOTS = 8) stream past L2
// (evict-first); half-sector flushes (SLOTS = 4) keep normal L2 priority so
// the sector's first half is still resident when its second half arrives.
template <int SLOTS>
__device__ __forceinline__ void st_row16(uint4* d, uint4 v)
{
    if constexpr (SLOTS == 8)
        __stcs(d, v);
    else
        __stcg(d, v);
}

// Write slots [k_lo, k_hi] of every real row of this thread's group.
//   row0: address of instance 32g's row; col: byte column of slot k_lo.
// Full segments go out as SLOTS/4 16 B stores (or 8 B stores when rows are only
// 8 B aligned, e.g. the paper's 4416-clock rows of 552 B); partial segments at
// item boundaries word by word.
template <int SLOTS = 8>
__device__ __forceinline__ void rowmajor_store(const uint32_t* os, uint8_t* row0, uint64_t row_bytes,
                                               uint32_t nvalid, uint32_t k_lo, uint32_t k_hi, uint64_t col)
{
    static_assert(SLOTS == 4 || SLOTS == 8, "SLOTS must be 4 or 8");
    uint8_t* p = row0 + col;
    const uint64_t align = reinterpret_cast<uintptr_t>(p) | row_bytes;
    if (k_lo == 0 && k_hi == SLOTS - 1 && (align & 15) == 0 && nvalid == 32) {
        // all shared-memory loads of RB rows first, then their stores, so a
        // lone warp does not wait out each load -> store latency per row.  The
        // batch is 16 registers: more and ptxas spills MICKEY's state words
        // inside the clock loop (it allocates the flush and the loop jointly)
        constexpr int RB = 16 / SLOTS;
#pragma unroll 1
        for (uint32_t q0 = 0; q0 < 32; q0 += RB) {
            uint32_t v[RB][SLOTS];
#pragma unroll
            for (int r = 0; r < RB; ++r)
#pragma unroll
                for (int k = 0; k < SLOTS; ++k) v[r][k] = os[((q0 + r) * SLOTS + k) * 32];
#pragma unroll
            for (int r = 0; r < RB; ++r) {
                uint4* d = reinterpret_cast<uint4*>(p + (q0 + r) * row_bytes);
#pragma unroll
                for (int k = 0; k < SLOTS; k += 4)
                    st_row16<SLOTS>(d + k / 4, make_uint4(v[r][k], v[r][k + 1], v[r][k + 2], v[r][k + 3]));
            }
        }
    } else if (k_lo == 0 && k_hi == SLOTS - 1 && (align & 15) == 0) {
#pragma unroll 4
        for (uint32_t q = 0; q < nvalid; ++q) {
            const uint32_t* src = os + q * SLOTS * 32;
            uint4* d = reinterpret_cast<uint4*>(p + q * row_bytes);
#pragma unroll
            for (int k = 0; k < SLOTS; k += 4)
                st_row16<SLOTS>(d + k / 4, make_uint4(src[k * 32], src[(k + 1) * 32], src[(k + 2) * 32],
                                                      src[(k + 3) * 32]));
        }
    } else if (k_lo == 0 && k_hi == SLOTS - 1 && (align & 7) == 0) {
#pragma unroll 4
        for (uint32_t q = 0; q < nvalid; ++q) {
            const uint32_t* src = os + q * SLOTS * 32;
            uint2* d = reinterpret_cast<uint2*>(p + q * row_bytes);
#pragma unroll
            for (int k = 0; k < SLOTS; k += 2) __stcs(d + k / 2, make_uint2(src[k * 32], src[(k + 1) * 32]));
        }
    } else {
        for (uint32_t q = 0; q < nvalid; ++q)
            for (uint32_t k = k_lo; k <= k_hi; ++k)
                __stcs(reinterpret_cast<uint32_t*>(p + q * row_bytes + (k - k_lo) * 4), os[(q * SLOTS + k) * 32]);
    }
}

// ---------------------------------------------------------------------------
// ROW_MAJOR staging in tensor memory (sm_100a TMEM, 128 lanes x 512 columns x
// 32 bit per SM).  Nothing here is a matrix product: TMEM is used as a plain
// per-thread staging buffer, because the whole-sector row buffer (32 rows x 8
// slots per thread = 32 KB per warp) does not fit twice per SMSP in shared
// memory, and half-sector flushes make L2 fetch and re-evict sectors (ncu:
// 13 GB of DRAM reads and 2x the writes for 8.6 GB of Grain keystream).  Warp
// w of a 4-warp CTA owns TMEM lanes 32(w%4)..+31 (its lane quarter); thread t
// stores row q's word for slot k at column q*8 + k of lane 32(w%4)+t, so a
// flush reads two rows' 8 slots with one 16-column load (16 registers).  Each
// CTA allocates 256 columns, so two CTAs (two clock-loop warps per SMSP) fit.
// ---------------------------------------------------------------------------
constexpr uint32_t TMEM_COLS = 256;

// dbl: 512 columns (two staging buffers; one CTA per SM, see KsArgs::tmem_dbl)
__device__ __forceinline__ uint32_t tmem_alloc_cta(uint32_t* s_base, bool dbl = false)
{
    if ((threadIdx.x >> 5) == 0) {
        const uint32_t sb = static_cast<uint32_t>(__cvta_generic_to_shared(s_base));
        if (dbl)
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(sb), "n"(2 * TMEM_COLS)
                         : "memory");
        else
            asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(sb), "n"(TMEM_COLS)
                         : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    return *reinterpret_cast<volatile uint32_t*>(s_base);
}

__device__ __forceinline__ void tmem_dealloc_cta(uint32_t base, bool dbl = false)
{
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if ((threadIdx.x >> 5) == 0) {
        if (dbl)
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(base), "n"(2 * TMEM_COLS)
                         : "memory");
        else
            asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(base), "n"(TMEM_COLS)
                         : "memory");
    }
}

// column taddr + OFF of this thread's lane <- v (one uniform base register,
// immediate column offsets: STTM tmem[UR + imm])
template <int OFF>
__device__ __forceinline__ void tmem_st1(uint32_t taddr, uint32_t v)
{
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0+%2], {%1};" ::"r"(taddr), "r"(v), "n"(OFF) : "memory");
}
// A TMEM address as a warp-uniform value: ptxas then keeps it in one uniform
// register and folds the column offsets into the STTMs (STTM tmem[UR+imm]);
// from a per-thread register it emitted one R2UR per STTM (32 per 32-clock
// block).
__device__ __forceinline__ uint32_t tmem_uniform(uint32_t taddr) { return __shfl_sync(0xFFFFFFFFu, taddr, 0); }

template <int H, int RS, int... Q>
__device__ __forceinline__ void tmem_st_rows(uint32_t base, const uint32_t (&x)[16], std::integer_sequence<int, Q...>)
{
    (tmem_st1<(16 * H + Q) * RS>(base, x[Q]), ...);
}

// v[0..15] <- 16 consecutive columns of this thread's lane (load + wait in one
// asm block, so no use of v can be scheduled before the data has arrived)
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16])
{
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15}, [%16];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr)
        : "memory");
}

__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// Transpose 32 z words held in registers and park the row words of slot k in
// TMEM columns q*RS + k (tm = this warp's lane-quarter base address; RS = 8
// slots per row, or 16 for the 64 B staging, where k is already the permuted
// column wide_col(slot)).
template <bool MSB_FIRST, int RS = 8>
__device__ __forceinline__ void rowmajor_transpose_tmem(const uint32_t (&z)[32], uint32_t tm, uint32_t k)
{
    constexpr int X = MSB_FIRST ? 7 : 0;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t x[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) x[q] = __byte_perm(z[q ^ X], z[(q + 16) ^ X], h == 0 ? 0x5410 : 0x7632);
        bt_transpose16(x);
        if (h == 0)
            tmem_st_rows<0, RS>(tmem_uniform(tm + k), x, std::make_integer_sequence<int, 16>{});
        else
            tmem_st_rows<1, RS>(tmem_uniform(tm + k), x, std::make_integer_sequence<int, 16>{});
    }
}
// The same from 32 z words staged in shared memory ([t][lane], zs = lane's column).
template <bool MSB_FIRST, int RS = 8>
__device__ __forceinline__ void rowmajor_transpose_smem_tmem(const uint32_t* zs, uint32_t tm, uint32_t k)
{
    constexpr int X = MSB_FIRST ? 7 : 0;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t x[16];
#pragma unroll
        for (int q = 0; q < 16; ++q)
            x[q] = __byte_perm(zs[(q ^ X) * 32], zs[((q + 16) ^ X) * 32], h == 0 ? 0x5410 : 0x7632);
        bt_transpose16(x);
        if (h == 0)
            tmem_st_rows<0, RS>(tmem_uniform(tm + k), x, std::make_integer_sequence<int, 16>{});
        else
            tmem_st_rows<1, RS>(tmem_uniform(tm + k), x, std::make_integer_sequence<int, 16>{});
    }
}

// The same from the writer-warp kernels' lane-major z block (rowmajor_ws.cuh
// ws::ZP): zl = this thread's 32 words (clock t at zl[t], 16 B aligned), read
// with 8 LDS.128 once for both 16-row halves.
template <bool MSB_FIRST, int RS>
__device__ __forceinline__ void rowmajor_transpose_lanes_tmem(const uint32_t* zl, uint32_t tm, uint32_t k)
{
    constexpr int X = MSB_FIRST ? 7 : 0;
    const uint32_t tmb = tmem_uniform(tm + k);
    uint32_t w[32];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        const uint4 v = *reinterpret_cast<const uint4*>(zl + 4 * i);
        w[4 * i] = v.x;
        w[4 * i + 1] = v.y;
        w[4 * i + 2] = v.z;
        w[4 * i + 3] = v.w;
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t x[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) x[q] = __byte_perm(w[q ^ X], w[(q + 16) ^ X], h == 0 ? 0x5410 : 0x7632);
        bt_transpose16(x);
        if (h == 0)
            tmem_st_rows<0, RS>(tmb, x, std::make_integer_sequence<int, 16>{});
        else
            tmem_st_rows<1, RS>(tmb, x, std::make_integer_sequence<int, 16>{});
    }
}

// Two consecutive blocks of the same rows (slots k, k + 1 at adjacent
// columns, k even under wide_col): both transposes interleaved (twice the
// independent work for a lone writer warp) and each row's two words written
// by one tcgen05.st.32x32b.x2 -- 32 instead of 64 STTM per pair (ptxas also
// emitted one R2UR per STTM).
template <int OFF>
__device__ __forceinline__ void tmem_st2(uint32_t taddr, uint32_t v0, uint32_t v1)
{
    asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0+%3], {%1, %2};" ::"r"(taddr), "r"(v0), "r"(v1), "n"(OFF)
                 : "memory");
}
template <int H, int RS, int... Q>
__device__ __forceinline__ void tmem_st_rows2(uint32_t base, const uint32_t (&x0)[16], const uint32_t (&x1)[16],
                                              std::integer_sequence<int, Q...>)
{
    (tmem_st2<(16 * H + Q) * RS>(base, x0[Q], x1[Q]), ...);
}
template <bool MSB_FIRST, int RS>
__device__ __forceinline__ void rowmajor_transpose_lanes_tmem2(const uint32_t* zl0, const uint32_t* zl1, uint32_t tm,
                                                               uint32_t k)
{
    constexpr int X = MSB_FIRST ? 7 : 0;
    uint32_t w0[32], w1[32];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        const uint4 v = *reinterpret_cast<const uint4*>(zl0 + 4 * i);
        const uint4 u = *reinterpret_cast<const uint4*>(zl1 + 4 * i);
        w0[4 * i] = v.x, w0[4 * i + 1] = v.y, w0[4 * i + 2] = v.z, w0[4 * i + 3] = v.w;
        w1[4 * i] = u.x, w1[4 * i + 1] = u.y, w1[4 * i + 2] = u.z, w1[4 * i + 3] = u.w;
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        uint32_t x0[16], x1[16];
#pragma unroll
        for (int q = 0; q < 16; ++q) {
            x0[q] = __byte_perm(w0[q ^ X], w0[(q + 16) ^ X], h == 0 ? 0x5410 : 0x7632);
            x1[q] = __byte_perm(w1[q ^ X], w1[(q + 16) ^ X], h == 0 ? 0x5410 : 0x7632);
        }
        bt_transpose16(x0);
        bt_transpose16(x1);
        if (h == 0)
            tmem_st_rows2<0, RS>(tmem_uniform(tm + k), x0, x1, std::make_integer_sequence<int, 16>{});
        else
            tmem_st_rows2<1, RS>(tmem_uniform(tm + k), x0, x1, std::make_integer_sequence<int, 16>{});
    }
}

// Flush slots [k_lo, k_hi] of every real row from TMEM (rowmajor_store's
// contract).  The loads are warp-collective, so every lane runs all of them;
// the per-lane row count only predicates the global stores.
__device__ __forceinline__ void rowmajor_store_tmem(uint32_t tm, uint8_t* row0, uint64_t row_bytes, uint32_t nvalid,
                                                    uint32_t k_lo, uint32_t k_hi, uint64_t col)
{
    tmem_wait_st();
    uint8_t* p = row0 + col;
    const uint64_t align = reinterpret_cast<uintptr_t>(p) | row_bytes;
    const bool full = k_lo == 0 && k_hi == 7;
#pragma unroll 1
    for (uint32_t q0 = 0; q0 < 32; q0 += 2) {
        uint32_t v[16];  // row q0 slots 0..7, row q0+1 slots 0..7
        tmem_ld16(tm + q0 * 8, v);
#pragma unroll
        for (int r = 0; r < 2; ++r) {
            if (q0 + r >= nvalid) continue;
            const uint32_t* w = v + 8 * r;
            uint8_t* d = p + (q0 + r) * row_bytes;
            if (full && (align & 15) == 0) {
                __stcs(reinterpret_cast<uint4*>(d), make_uint4(w[0], w[1], w[2], w[3]));
                __stcs(reinterpret_cast<uint4*>(d) + 1, make_uint4(w[4], w[5], w[6], w[7]));
            } else if (full && (align & 7) == 0) {
#pragma unroll
                for (int k = 0; k < 8; k += 2) __stcs(reinterpret_cast<uint2*>(d) + k / 2, make_uint2(w[k], w[k + 1]));
            } else {
#pragma unroll
                for (int k = 0; k < 8; ++k)
                    if (uint32_t(k) >= k_lo && uint32_t(k) <= k_hi)
                        __stcs(reinterpret_cast<uint32_t*>(d) + (k - k_lo), w[k]);
            }
        }
    }
}

__device__ __forceinline__ uint32_t tid_volatile()
{
    uint32_t v;
    asm volatile("mov.u32 %0, %%tid.x;" : "=r"(v));
    return v;
}

__device__ __forceinline__ uint32_t laneid_volatile()
{
    uint32_t v;
    asm volatile("mov.u32 %0, %%laneid;" : "=r"(v));
    return v;
}
// threadIdx.x >> 5 re-read from the special register (S2R) where it is used,
// so that ptxas cannot keep it -- or addresses derived from it -- live across
// a register-saturated clock loop (it spilled them: one local-memory reload on
// the critical path of every 32-clock block)
__device__ __forceinline__ uint32_t warp_volatile()
{
    uint32_t v;
    asm volatile("mov.u32 %0, %%tid.x;" : "=r"(v));
    return v >> 5;
}

// p + d as one IMAD.WIDE.U32 (FMA pipe) instead of IADD3 + IADD3.X (ALU);
// d < 2^32 (row strides)
__device__ __forceinline__ uint8_t* add_fma(uint8_t* p, uint64_t d)
{
    uint64_t r;
    asm("mad.wide.u32 %0, %1, 1, %2;" : "=l"(r) : "r"(uint32_t(d)), "l"(reinterpret_cast<uint64_t>(p)));
    return reinterpret_cast<uint8_t*>(r);
}

__device__ __forceinline__ uint64_t l2_evict_last_policy()
{
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// WS_EXPERIMENT_NO_STG (measurement builds only, no output): the hinted
// flush stores keep their operands live but issue nothing, which separates
// the flush's TMEM read-back / address work from its DRAM writes
#ifdef WS_EXPERIMENT_NO_STG
#define BSK_NO_STG_RETURN(...) do { asm volatile("" ::__VA_ARGS__); return; } while (0)
#else
#define BSK_NO_STG_RETURN(...) do { } while (0)
#endif
__device__ __forceinline__ void st128_hint(uint8_t* p, uint32_t a, uint32_t b, uint32_t c, uint32_t d, uint64_t pol)
{
    BSK_NO_STG_RETURN("l"(p), "r"(a), "r"(b), "r"(c), "r"(d));
    asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p), "r"(a), "r"(b), "r"(c),
                 "r"(d), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void st64_hint(uint8_t* p, uint32_t a, uint32_t b, uint64_t pol)
{
    BSK_NO_STG_RETURN("l"(p), "r"(a), "r"(b));
    asm volatile("st.global.L2::cache_hint.v2.u32 [%0], {%1, %2}, %3;" ::"l"(p), "r"(a), "r"(b), "l"(pol) : "memory");
}
// 8 B sector-flush store: evict-first (streaming), or with an L2 evict_last
// hint (pol != 0) so a row's next sector finds its 128 B line still resident
__device__ __forceinline__ void st_sector8(uint8_t* p, uint32_t a, uint32_t b, uint64_t pol)
{
    if (pol)
        st64_hint(p, a, b, pol);
    else
        __stcs(reinterpret_cast<uint2*>(p), make_uint2(a, b));
}

// v[0..15] <- tcgen05.ld.16x256b.x4 at taddr: thread t receives, for repeat
// i = 0..3 (columns +8i), TMEM lane base+t/4 columns 2(t%4), 2(t%4)+1 in
// v[4i], v[4i+1] and lane base+8+t/4 (same columns) in v[4i+2], v[4i+3]
// (fragment layout measured on the B200: tools/microbench/tmem_layout.cu).
__device__ __forceinline__ void tmem_ld16x256b_x4(uint32_t taddr, uint32_t (&v)[16])
{
    asm volatile(
        "tcgen05.ld.sync.aligned.16x256b.x4.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15}, [%16];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr)
        : "memory");
}

// The same for 8 repeats (64 columns, 32 registers): two row pairs per
// tcgen05.wait::ld, so the flush loops pay the TMEM load latency once per four
// rows instead of once per two (ncu: the writer warp's flush loop waited on
// the x4 load's scoreboard for ~60% of its samples).
__device__ __forceinline__ void tmem_ld16x256b_x8(uint32_t taddr, uint32_t (&v)[32])
{
    asm volatile(
        "tcgen05.ld.sync.aligned.16x256b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
        "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];\n\t"
        "tcgen05.wait::ld.sync.aligned;"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15]),
          "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]),
          "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
        : "r"(taddr)
        : "memory");
}

// Whole-sector flush (slots 0..7 of every row, 8 B aligned rows) read back
// with the 16x256b shape: four consecutive threads receive one TMEM lane's
// (= one instance row's) 32 B sector, so each 8 B store instruction writes 8
// complete sectors (8 L1 wavefronts) instead of 32 half sectors from 32
// threads' own rows (the 32x32b read-back: 2048 wavefronts and 2048 partial
// sector writes per flush, 22% of Grain's ROW_MAJOR time in ncu's stall
// samples).  row0s / nvalids: this warp's per-thread row bases and row counts
// (shared memory, indexed by the thread = TMEM lane that computed them).
__device__ __forceinline__ void rowmajor_store_tmem_sectors(uint32_t tm, uint8_t* const* row0s,
                                                            const uint32_t* nvalids, uint64_t row_bytes, uint64_t col,
                                                            bool l2last = false)
{
    tmem_wait_st();
    const uint64_t pol = l2last ? l2_evict_last_policy() : 0ull;
    const uint32_t t = laneid_volatile();
#pragma unroll 1
    for (uint32_t h = 0; h < 2; ++h) {
        const uint32_t la = 16 * h + (t >> 2), lb = la + 8;
        // running row pointers: 64-bit adds per row instead of multiplies
        uint8_t* pa = row0s[la] + col + 8 * (t & 3);
        uint8_t* pb = row0s[lb] + col + 8 * (t & 3);
        const uint32_t na = nvalids[la], nb = nvalids[lb];
        if (__all_sync(0xFFFFFFFFu, (na & nb) == 32)) {
            // every row real (all but the last warp-unit): no predicates, and
            // the row addresses advance on the FMA pipe (IMAD.WIDE) -- the
            // clock loop saturates the ALU pipe
#pragma unroll 1
            for (uint32_t q0 = 0; q0 < 32; q0 += 4) {
                uint32_t v[16];
                tmem_ld16x256b_x4(tm + ((16 * h) << 16) + q0 * 8, v);
#pragma unroll
                for (int i = 0; i < 4; ++i) {
                    st_sector8(pa, v[4 * i], v[4 * i + 1], pol);
                    st_sector8(pb, v[4 * i + 2], v[4 * i + 3], pol);
                    pa = add_fma(pa, row_bytes);
                    pb = add_fma(pb, row_bytes);
                }
            }
            continue;
        }
#pragma unroll 1
        for (uint32_t q0 = 0; q0 < 32; q0 += 4) {
            uint32_t v[16];
            tmem_ld16x256b_x4(tm + ((16 * h) << 16) + q0 * 8, v);
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                if (q0 + i < na) __stcs(reinterpret_cast<uint2*>(pa), make_uint2(v[4 * i], v[4 * i + 1]));
                if (q0 + i < nb) __stcs(reinterpret_cast<uint2*>(pb), make_uint2(v[4 * i + 2], v[4 * i + 3]));
                pa += row_bytes;
                pb += row_bytes;
            }
        }
    }
}

// ---------------------------------------------------------------------------
// TMA-store flush (ROW_MAJOR, TMEM staging).  The 16x256b read-back gives four
// threads one row's 32 B sector; instead of 128 scattered 8 B global stores
// per thread (whose address/data registers the next instructions must wait
// to reuse until the LSU has drained them -- ncu: long-scoreboard stalls on
// the flush's address adds, 12.6% of Grain's ROW_MAJOR time), each warp
// writes the sectors into a 16 KB shared-memory box and one lane issues TMA
// tensor stores, which move the 1024 scattered sectors asynchronously while
// the warp returns to its clock loop.
// Tensor map (bsrng.cu): dims {row_bytes, tma_groups, 32} with strides
// {32 row_bytes, row_bytes}, i.e. element (byte c, group g, q) = out[(32 g + q)
// * row_bytes + c]; box {32, 8, 32} = 8 groups x 32 instances x one 32 B
// sector, laid out in smem as [q][group][32 B] so a 16x256b fragment (8
// groups x 32 B for one q) is 256 contiguous bytes: conflict-free 8 B stores.
// ---------------------------------------------------------------------------
// Rows q in [q_lo, q_hi) (multiples of 4) of a whole-sector period, every
// row real and 8 B aligned (tmem_dbl's progressive flush): 16x256b read-back,
// unpredicated 8 B stores.
__device__ __forceinline__ void rowmajor_store_tmem_rows(uint32_t tm, uint8_t* const* row0s, uint64_t row_bytes,
                                                         uint64_t col, uint32_t q_lo, uint32_t q_hi, bool l2last = false)
{
    tmem_wait_st();
    const uint64_t pol = l2last ? l2_evict_last_policy() : 0ull;
    const uint32_t t = laneid_volatile();
#pragma unroll 1
    for (uint32_t h = 0; h < 2; ++h) {
        const uint32_t la = 16 * h + (t >> 2), lb = la + 8;
        uint8_t* pa = row0s[la] + col + 8 * (t & 3) + q_lo * row_bytes;
        uint8_t* pb = row0s[lb] + col + 8 * (t & 3) + q_lo * row_bytes;
#pragma unroll 1
        for (uint32_t q0 = q_lo; q0 < q_hi; q0 += 4) {
            uint32_t v[16];
            tmem_ld16x256b_x4(tm + ((16 * h) << 16) + q0 * 8, v);
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                st_sector8(pa, v[4 * i], v[4 * i + 1], pol);
                st_sector8(pb, v[4 * i + 2], v[4 * i + 3], pol);
                pa += row_bytes;
                pb += row_bytes;
            }
        }
    }
}

// ---------------------------------------------------------------------------
// 64 B staging ("wide": one clock-loop warp per SMSP owns all 512 TMEM
// columns of its lane quarter).  Row q's 16 slot words live at columns
// q*16 + wide_col(k), permuted so that the tcgen05.ld.16x256b read-back hands
// thread j = t%4 the slots 4j..4j+3 -- 16 contiguous bytes -- of the rows in
// TMEM lanes t/4 and t/4+8: every STG.128 writes 8 rows x 64 B.  Why 64 B:
// the flush_pattern microbenchmark (profiles/r2_flush_pattern.log) writes the
// kernels' output pattern (1024 rows per warp, one piece per row per flush)
// without compute: 32 B per row per flush reaches 1.4-1.8 TB/s, 64 B 2.9-3.6
// TB/s (DRAM page locality).  The stores carry an L2 evict_last hint (3.55 vs
// 2.93 TB/s at 64 B): a row's next piece lands on the same 128 B line.
// ---------------------------------------------------------------------------
__host__ __device__ constexpr uint32_t wide_col(uint32_t k)
{
    return 2 * (k >> 2) + (k & 1) + ((k & 2) ? 8 : 0);
}


// Whole 64 B flush (slots 0..15 of every row; rows 8 B aligned: 16 B
// aligned rows take one STG.128 per row piece, 8 B aligned ones -- e.g. the
// paper shape's 552 B rows -- two STG.64).  row0s / nvalids: this warp's
// per-thread row bases and real-row counts (smem).
__device__ __forceinline__ void st_piece16(uint8_t* p, uint32_t a, uint32_t b, uint32_t c, uint32_t d, uint64_t pol,
                                           bool a16)
{
    if (a16) {
        st128_hint(p, a, b, c, d, pol);
    } else {
        st64_hint(p, a, b, pol);
        st64_hint(p + 8, c, d, pol);
    }
}
__device__ __forceinline__ void rowmajor_store_tmem_wide(uint32_t tm, uint8_t* const* row0s, const uint32_t* nvalids,
                                                         uint64_t row_bytes, uint64_t col)
{
    tmem_wait_st();
    const uint32_t t = laneid_volatile();
    const uint64_t pol = l2_evict_last_policy();
    const bool a16 = ((row_bytes | col) & 15) == 0;
#pragma unroll 1
    for (uint32_t h = 0; h < 2; ++h) {
        const uint32_t la = 16 * h + (t >> 2), lb = la + 8;
        uint8_t* pa = row0s[la] + col + 16 * (t & 3);
        uint8_t* pb = row0s[lb] + col + 16 * (t & 3);
        const uint32_t na = nvalids[la], nb = nvalids[lb];
        if (a16 && __all_sync(0xFFFFFFFFu, (na & nb) == 32)) {
#pragma unroll 1
            for (uint32_t q = 0; q < 32; q += 4) {
                uint32_t v[32];  // rows q..q+3 (v[8r..8r+7]) of lanes la (v[8r+4i], +1) / lb (+2, +3)
                tmem_ld16x256b_x8(tm + ((16 * h) << 16) + q * 16, v);
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    st128_hint(pa, v[8 * r], v[8 * r + 1], v[8 * r + 4], v[8 * r + 5], pol);
                    st128_hint(pb, v[8 * r + 2], v[8 * r + 3], v[8 * r + 6], v[8 * r + 7], pol);
                    pa = add_fma(pa, row_bytes);
                    pb = add_fma(pb, row_bytes);
                }
            }
            continue;
        }
#pragma unroll 1
        for (uint32_t q = 0; q < 32; q += 4) {
            uint32_t v[32];
            tmem_ld16x256b_x8(tm + ((16 * h) << 16) + q * 16, v);
#pragma unroll
            for (int r = 0; r < 4; ++r) {
                if (q + r < na) st_piece16(pa, v[8 * r], v[8 * r + 1], v[8 * r + 4], v[8 * r + 5], pol, a16);
                if (q + r < nb) st_piece16(pb, v[8 * r + 2], v[8 * r + 3], v[8 * r + 6], v[8 * r + 7], pol, a16);
                pa += row_bytes;
                pb += row_bytes;
            }
        }
    }
}

__device__ __forceinline__ void st32_hint(uint8_t* p, uint32_t a, uint64_t pol)
{
    BSK_NO_STG_RETURN("l"(p), "r"(a));
    asm volatile("st.global.L2::cache_hint.u32 [%0], %1, %2;" ::"l"(p), "r"(a), "l"(pol) : "memory");
}
// Store the run of slots [m0, m1] (0 <= m0, m1 <= 3; empty if m0 > m1) of one
// row's 16 B piece w[0..3]; A = the address slot 0 of the piece would have.
// Widest aligned stores: 16 B for a whole 16 B aligned piece, else 8 B pairs
// on 8 B boundaries and 4 B singles (rows are at least 4 B aligned).
__device__ __forceinline__ void st_run4(uint8_t* A, uint32_t w0, uint32_t w1, uint32_t w2, uint32_t w3, int m0,
                                        int m1, uint64_t pol)
{
    const bool r0 = m0 <= 0 && 0 <= m1, r1 = m0 <= 1 && 1 <= m1, r2 = m0 <= 2 && 2 <= m1, r3 = m0 <= 3 && 3 <= m1;
    const uint32_t al = uint32_t(reinterpret_cast<uintptr_t>(A)) & 15u;
    if ((al & 7u) == 0) {
        if (r0 && r3 && al == 0) {
            st128_hint(A, w0, w1, w2, w3, pol);
            return;
        }
        if (r0 && r1) st64_hint(A, w0, w1, pol);
        else if (r0) st32_hint(A, w0, pol);
        else if (r1) st32_hint(A + 4, w1, pol);
        if (r2 && r3) st64_hint(A + 8, w2, w3, pol);
        else if (r2) st32_hint(A + 8, w2, pol);
        else if (r3) st32_hint(A + 12, w3, pol);
    } else {
        if (r0) st32_hint(A, w0, pol);
        if (r1 && r2 && (al & 7u) == 4u) st64_hint(A + 4, w1, w2, pol);
        else {
            if (r1) st32_hint(A + 4, w1, pol);
            if (r2) st32_hint(A + 8, w2, pol);
        }
        if (r3) st32_hint(A + 12, w3, pol);
    }
}

// Partial 64 B flush: slots [k_lo, k_hi] only (item boundaries that are not
// whole 512-clock periods, e.g. the paper shape's 4416 clocks = 8 periods + 10
// slots).  Same 16x256b read-back as the whole flush; thread j = t%4 holds
// slots 4j..4j+3 of its rows and stores the part of them inside [k_lo, k_hi]
// with the widest aligned stores (st_run4): the paper shape's closing 40 B
// leave as 8 B stores instead of one 4 B store per slot (this flush runs after
// the clock loop has ended, so it is the kernel's tail).
__device__ __forceinline__ void rowmajor_store_tmem_wide_partial(uint32_t tm, uint8_t* const* row0s,
                                                                 const uint32_t* nvalids, uint64_t row_bytes,
                                                                 uint32_t k_lo, uint32_t k_hi, uint64_t col)
{
    tmem_wait_st();
    const uint32_t t = laneid_volatile();
    const uint32_t j = t & 3u;
    const uint64_t pol = l2_evict_last_policy();
    // this thread's run [m0, m1] of slots 4j + m inside [k_lo, k_hi]
    const int lo = int(k_lo > 4 * j ? k_lo : 4 * j), hi = int(k_hi < 4 * j + 3 ? k_hi : 4 * j + 3);
    const int m0 = lo - int(4 * j), m1 = hi - int(4 * j);  // empty when lo > hi
    // A = address of slot 4j: piece start + (4j - k_lo) words (may precede it)
    const int64_t off = int64_t(col) + 4 * (int64_t(4 * j) - int64_t(k_lo));
#pragma unroll 1
    for (uint32_t h = 0; h < 2; ++h) {
        const uint32_t la = 16 * h + (t >> 2), lb = la + 8;
        uint8_t* pa = row0s[la] + off;
        uint8_t* pb = row0s[lb] + off;
        const uint32_t na = nvalids[la], nb = nvalids[lb];
#pragma unroll 1
        for (uint32_t q = 0; q < 32; q += 4) {
            uint32_t v[32];
            tmem_ld16x256b_x8(tm + ((16 * h) << 16) + q * 16, v);
            if (m0 <= m1) {
#pragma unroll
                for (int r = 0; r < 4; ++r) {
                    if (q + r < na) st_run4(pa, v[8 * r], v[8 * r + 1], v[8 * r + 4], v[8 * r + 5], m0, m1, pol);
                    if (q + r < nb) st_run4(pb, v[8 * r + 2], v[8 * r + 3], v[8 * r + 6], v[8 * r + 7], m0, m1, pol);
                    pa += row_bytes;
                    pb += row_bytes;
                }
            }
        }
    }
}

__device__ __forceinline__ uint32_t smem_addr_u32(const void* p)
{
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void bulk_wait_read_all() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void tma_store_3d_hint(const CUtensorMap* map, uint32_t src, int c0, int c1, int c2,
                                                  uint64_t pol)
{
    asm volatile(
        "cp.async.bulk.tensor.3d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%2, %3, %4}], [%1], %5;" ::"l"(
            reinterpret_cast<uint64_t>(map)),
        "r"(src), "r"(c0), "r"(c1), "r"(c2), "l"(pol)
        : "memory");
}
__device__ __forceinline__ void tma_store_3d(const CUtensorMap* map, uint32_t src, int c0, int c1, int c2)
{
    asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%2, %3, %4}], [%1];" ::"l"(
                     reinterpret_cast<uint64_t>(map)),
                 "r"(src), "r"(c0), "r"(c1), "r"(c2)
                 : "memory");
}
constexpr int TMA_BUF_WORDS = 4096;  // 16 KB per warp: two 8 KB boxes

// One half of a TMA flush: TMEM lanes 16h..16h+15 (groups g_w0 + 16h ..
// +15, two 8-group boxes).  The second half of a flush is deferred to the
// start of the warp's next 32-clock block (before that block's transpose
// overwrites slot 0), so the TMA engine has a block's worth of clocks to read
// the first half's boxes out of the 16 KB buffer; waiting for those reads
// right away cost 8.6% of Grain's ROW_MAJOR time (ncu: BSYNC after lane 0's
// cp.async.bulk.wait_group.read).
__device__ __forceinline__ void tma_flush_half(uint32_t tm, uint32_t* buf, const CUtensorMap* map, uint64_t g_w0,
                                               uint64_t col, uint32_t h, bool l2last = false)
{
    const uint32_t t = laneid_volatile();
    const uint32_t sb = smem_addr_u32(buf);
    const uint32_t off_t = (t >> 2) * 32 + (t & 3) * 8;
    if (t == 0) bulk_wait_read_all();  // the previous boxes have left the buffer
    __syncwarp();
#pragma unroll 1
    for (uint32_t q0 = 0; q0 < 32; q0 += 4) {
        uint32_t v[16];
        tmem_ld16x256b_x4(tm + ((16 * h) << 16) + q0 * 8, v);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const uint32_t o = sb + (q0 + i) * 256 + off_t;
            asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"(o), "r"(v[4 * i]), "r"(v[4 * i + 1]) : "memory");
            asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"(o + 8192), "r"(v[4 * i + 2]), "r"(v[4 * i + 3])
                         : "memory");
        }
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic-proxy writes -> TMA reads
    __syncwarp();
    if (t == 0) {
        const int g = int(g_w0 + 16 * h);
        if (l2last) {
            const uint64_t pol = l2_evict_last_policy();
            tma_store_3d_hint(map, sb, int(col), g, 0, pol);
            tma_store_3d_hint(map, sb + 8192, int(col), g + 8, 0, pol);
        } else {
            tma_store_3d(map, sb, int(col), g, 0);
            tma_store_3d(map, sb + 8192, int(col), g + 8, 0);
        }
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
}

// Fetch the next work item for this warp into smem (persistent mode).
__device__ __forceinline__ void next_item(const KsArgs& a, volatile uint32_t* slot)
{
    __syncwarp();
    if (laneid_volatile() == 0) *slot = atomicAdd(a.ticket, 1u);
    __syncwarp();
}

// SLOTS: row-segment slots staged in smem (8 or 4); TMEM: stage in tensor
// memory instead (8 slots, no smem for rows); ZREG: see rm_warp_words.
// DBL: double-buffered TMEM staging (KsArgs::tmem_dbl), a separate instance so
// the single-buffer kernel carries none of its code (measured: 0.3%)
// WIDE: 64 B TMEM staging per row (one CTA per SM, all 512 columns, 16 slots).
template <class C, int LAYOUT, int U, int BLOCK, int SLOTS = 8, bool ZREG = true, bool TMEM = false, bool DBL = false,
          bool WIDE = false>
__global__ void __launch_bounds__(BLOCK) keystream_kernel(const __grid_constant__ KsArgs a)
{
    static_assert(32 % U == 0, "U must divide 32");
    constexpr int KB = ks_block<C, U>();  // clocks per cipher schedule block
    static_assert(U % KB == 0, "the loop body must hold whole schedule blocks");
    constexpr int NW = BLOCK / 32;
    // ROW_MAJOR only: NW * rm_warp_words(U, SLOTS, ZREG) (TMEM: NW * ZS_WORDS, none with ZREG),
    // then NW * TMA_BUF_WORDS when a.use_tma
    extern __shared__ __align__(1024) uint32_t rm_smem[];
    __shared__ uint8_t* s_row0[LAYOUT == L_ROW_MAJOR ? BLOCK : 1];
    __shared__ uint32_t s_nvalid[LAYOUT == L_ROW_MAJOR ? BLOCK : 1];
    __shared__ uint64_t s_b0[LAYOUT == L_ROW_MAJOR ? NW : 1];
    __shared__ uint32_t s_nblk[LAYOUT == L_ROW_MAJOR ? NW : 1];
    // TMA flush whose second half is pending (col + 1, 0 = none) and its first group
    __shared__ uint64_t s_pend_col[LAYOUT == L_ROW_MAJOR && TMEM ? NW : 1];
    __shared__ uint64_t s_pend_g[LAYOUT == L_ROW_MAJOR && TMEM ? NW : 1];
    // tmem_dbl: the previous sector period still being flushed (col + 1, 0 = none)
    __shared__ uint64_t s_pdbl_col[LAYOUT == L_ROW_MAJOR && TMEM ? NW : 1];
    __shared__ uint32_t s_item[NW];
    // Only `s_item` (smem) and the loop counters survive a clock loop; every
    // other per-item value is re-derived afterwards, so the 200 state words
    // plus temporaries fit in 255 registers without spilling.
    volatile uint32_t* slot = s_item + (threadIdx.x >> 5);
    // TMEM staging: the CTA's allocation base lives in smem and each use
    // re-derives this warp's lane-quarter address (no register held across
    // the clock loop)
    __shared__ uint32_t s_tmem;
    if constexpr (LAYOUT == L_ROW_MAJOR && TMEM) {
        static_assert(BLOCK == 128, "TMEM staging maps warp w to lane quarter w");
        static_assert(!(DBL && WIDE), "one 512-column TMEM use at a time");
        (void)tmem_alloc_cta(&s_tmem, DBL || WIDE);
        if (laneid_volatile() == 0) s_pend_col[threadIdx.x >> 5] = s_pdbl_col[threadIdx.x >> 5] = 0;
    }
    // tmem_dbl: sector period B >> 3 stages into buffer (B >> 3) & 1
    auto dbl_off = [&](uint64_t B) -> uint32_t { return DBL ? uint32_t((B >> 3) & 1) * TMEM_COLS : 0u; };
    auto tm_addr = [&]() {
        return *reinterpret_cast<volatile uint32_t*>(&s_tmem) + ((threadIdx.x >> 5) << 21);
    };
    auto tma_buf = [&]() {
        return rm_smem + NW * (U == 32 && ZREG ? 0 : ZS_WORDS) + (tid_volatile() >> 5) * TMA_BUF_WORDS;
    };
    // issue the deferred second half of the previous block's TMA flush
    auto tma_pending = [&]() {
        if constexpr (LAYOUT == L_ROW_MAJOR && TMEM) {
            const uint32_t wq = tid_volatile() >> 5;
            const uint64_t pc = *reinterpret_cast<volatile uint64_t*>(&s_pend_col[wq]);
            if (pc) {
                tma_flush_half(tm_addr(), tma_buf(), &a.tmap, *reinterpret_cast<volatile uint64_t*>(&s_pend_g[wq]),
                               pc - 1, 1, a.l2last);
                __syncwarp();
                if (laneid_volatile() == 0) s_pend_col[wq] = 0;
                __syncwarp();
            }
        }
    };
    if (a.persistent)
        next_item(a, slot);
    else if (laneid_volatile() == 0)
        *slot = (blockIdx.x * BLOCK + threadIdx.x) >> 5;
    __syncwarp();

    const uint64_t total = a.units * a.nseg;
    for (;;) {
        uint64_t item = *slot;
        if (item >= total) break;
        uint32_t lane = laneid_volatile();
        uint64_t seg = item / a.units;
        uint64_t w = item - seg * a.units;
        uint64_t g = w * 32u + lane;
        if (seg > 0) {
            if (lane == 0)
            {
                uint32_t spins = 0;
                while (ld_acquire(a.flags + w) < seg) {
                    __nanosleep(256);
                    ++spins;
                }
                if (a.dbg) {
                    atomicAdd(a.dbg + 0, 1ull);
                    if (spins) atomicAdd(a.dbg + 1, 1ull);
                    atomicAdd(a.dbg + 2, (unsigned long long)spins);
                }
            }
            __syncwarp();
            (void)ld_acquire(a.flags + w);
        }
        const uint64_t clk_begin = seg * a.seg_clocks;
        const uint64_t left = a.nclocks - clk_begin;
        const uint32_t nclk = uint32_t(left < a.seg_clocks ? left : a.seg_clocks);

        C c;
        c.load(a.state, a.Gp, g);
        uint32_t acc = 0;
        if (LAYOUT == L_CHECKSUM && seg > 0) acc = __ldcg(a.state + uint64_t(C::NSTATE) * a.Gp + g);

        if (LAYOUT == L_CHECKSUM) {
            uint32_t nrem = nclk;
            if constexpr (ks_u_big<C>::value > 0) {
                constexpr int UB = ks_u_big<C>::value;
                static_assert(KB == 1, "long consume bodies only for unphased ciphers");
                // the remainder must be whole U-clock iterations: split at a
                // multiple of lcm(UB, 32)
                constexpr uint32_t L = UB % 32 == 0 ? UB : (UB % 16 == 0 ? 2 * UB : 4 * UB);
                nrem = nclk % L;
#pragma unroll 1
                for (uint32_t it = (nclk - nrem) / UB; it != 0; --it) {
                    if constexpr (ks_period<C>::value) {
                        c.consume_period(acc);
                    } else {
                        static_for<UB>([&](auto) {
                            acc = ks_z_acc<0, 1>(c, acc);
                            ks_clock<0, 1>(c);
                        });
                    }
                }
            }
#pragma unroll 1
            for (uint32_t it = nrem / U; it != 0; --it) {
                static_for<U>([&](auto u) {
                    constexpr int J = decltype(u)::value % KB;
                    acc = ks_z_acc<J, KB>(c, acc);
                    ks_clock<J, KB>(c);
                });
            }
        } else if (LAYOUT == L_SLICED) {
            const uint32_t m = lane_mask(a, g);
            // padding groups (g >= G) write to a private scratch word instead of
            // being predicated off, so the loop body has no branches
            uint32_t* o = g < a.G ? static_cast<uint32_t*>(a.out) + clk_begin * a.G + g : a.scratch + lane;
            const uint64_t stride = g < a.G ? a.G : 0;
#pragma unroll 1
            for (uint32_t it = nclk / U; it != 0; --it) {
                static_for<U>([&](auto u) {
                    constexpr int J = decltype(u)::value % KB;
                    __stcs(o, ks_z<J, KB>(c) & m);
                    o += stride;
                    ks_clock<J, KB>(c);
                });
            }
        } else {  // ROW_MAJOR
            const uint64_t first = g * 32u;
            const uint32_t nvalid = first >= a.n ? 0u : uint32_t(a.n - first < 32 ? a.n - first : 32);
            s_row0[threadIdx.x] = static_cast<uint8_t*>(a.out) + (nvalid ? first : 0) * a.row_bytes;
            s_nvalid[threadIdx.x] = nvalid;
            // per-warp block context in smem: only `blk` stays in a register
            // across the clock loop (MICKEY's 200 state words leave ~40)
            if (lane == 0) {
                s_b0[threadIdx.x >> 5] = clk_begin >> 5;  // call-relative index of the item's first block
                s_nblk[threadIdx.x >> 5] = uint32_t(nclk >> 5);
            }
            __syncwarp();
            constexpr uint32_t NSLOT = TMEM ? (WIDE ? 16 : 8) : SLOTS;
            constexpr int RS = WIDE ? 16 : 8;  // TMEM columns per row
            // TMEM column of slot k (WIDE: permuted for the 16x256b read-back)
            auto tcol = [&](uint64_t B, uint32_t k) { return WIDE ? wide_col(k) : dbl_off(B) + k; };
            constexpr int WW = TMEM ? ZS_WORDS : rm_warp_words(U, SLOTS, ZREG);
            // re-derived after every clock loop from non-CSE-able special registers
            auto zs_ptr = [&]() { return rm_smem + (tid_volatile() >> 5) * WW + laneid_volatile(); };
            auto os_ptr = [&]() { return zs_ptr() + (U == 32 && ZREG ? 0 : ZS_WORDS); };
#pragma unroll 1
            for (uint32_t blk = 0;; ++blk) {
                const uint32_t nblk = *reinterpret_cast<volatile uint32_t*>(&s_nblk[tid_volatile() >> 5]);
                if (blk >= nblk) break;
                if constexpr (U == 32 && ZREG) {
                    // one 32-clock block per iteration: keep the z words in
                    // registers and transpose them there (no z staging in smem)
                    uint32_t zr[32];
                    static_for<32>([&](auto u) {
                        constexpr int J = decltype(u)::value % KB;
                        zr[decltype(u)::value] = ks_z<J, KB>(c);
                        ks_clock<J, KB>(c);
                    });
                    const uint64_t B = *reinterpret_cast<volatile uint64_t*>(&s_b0[tid_volatile() >> 5]) + blk;
                    const uint32_t k = uint32_t(B & (NSLOT - 1));
                    tma_pending();
                    if constexpr (TMEM)
                        rowmajor_transpose_tmem<C::MSB_FIRST, RS>(zr, tm_addr(), tcol(B, k));
                    else
                        rowmajor_transpose_regs<C::MSB_FIRST, SLOTS>(zr, os_ptr(), k);
                } else {
                    uint32_t* zs = zs_ptr();
#pragma unroll 1
                    for (uint32_t kk = 0; kk < 32; kk += U) {
                        static_for<U>([&](auto u) {
                            constexpr int J = decltype(u)::value % KB;
                            zs[(kk + decltype(u)::value) * 32] = ks_z<J, KB>(c);
                            ks_clock<J, KB>(c);
                        });
                    }
                    const uint64_t B = *reinterpret_cast<volatile uint64_t*>(&s_b0[tid_volatile() >> 5]) + blk;
                    const uint32_t k = uint32_t(B & (NSLOT - 1));
                    tma_pending();
                    if constexpr (TMEM)
                        rowmajor_transpose_smem_tmem<C::MSB_FIRST, RS>(zs_ptr(), tm_addr(), tcol(B, k));
                    else
                        rowmajor_transpose<C::MSB_FIRST, SLOTS>(zs_ptr(), os_ptr(), k);
                }
                const uint64_t B = *reinterpret_cast<volatile uint64_t*>(&s_b0[tid_volatile() >> 5]) + blk;
                const uint32_t k = uint32_t(B & (NSLOT - 1));
                if constexpr (TMEM) {
                    // tmem_dbl: 4 rows of the previous period per block (the rest
                    // at the item's last block), from the other buffer
                    if constexpr (DBL) {
                        const uint32_t wq = tid_volatile() >> 5;
                        const uint64_t pc = *reinterpret_cast<volatile uint64_t*>(&s_pdbl_col[wq]);
                        if (pc) {
                            const uint32_t q_hi = blk + 1 == nblk ? 32u : 4 * k + 4;
                            rowmajor_store_tmem_rows(tm_addr() + (dbl_off(B) ^ TMEM_COLS), s_row0 + wq * 32,
                                                     a.row_bytes, pc - 1, 4 * k, q_hi, a.l2last);
                            if (q_hi == 32) {
                                __syncwarp();
                                if (laneid_volatile() == 0) s_pdbl_col[wq] = 0;
                                __syncwarp();
                            }
                        }
                    }
                }
                if (k == NSLOT - 1 || blk + 1 == nblk) {
                    const uint32_t k_lo = k - (blk < k ? blk : k);
                    const uint32_t t = tid_volatile();
                    const uint64_t col = (B - (k - k_lo)) * 4;
                    if constexpr (TMEM) {
                        const uint64_t g_w0 = (*slot % a.units) * 32u;  // the warp's first group
                        const bool full_real = __all_sync(0xFFFFFFFFu, s_nvalid[t] == 32);
                        if constexpr (WIDE) {
                            (void)full_real;
                            (void)g_w0;
                            if (k_lo == 0 && k == NSLOT - 1 && ((a.row_bytes | col) & 7) == 0 &&
                                a.row_bytes < (1ull << 32))
                                rowmajor_store_tmem_wide(tm_addr(), s_row0 + (t & ~31u), s_nvalid + (t & ~31u),
                                                         a.row_bytes, col);
                            else
                                rowmajor_store_tmem_wide_partial(tm_addr(), s_row0 + (t & ~31u),
                                                                 s_nvalid + (t & ~31u), a.row_bytes, k_lo, k, col);
                        } else if (DBL && k_lo == 0 && k == 7 && blk + 1 < nblk && full_real &&
                            ((a.row_bytes | col) & 7) == 0) {
                            // flushed during the next period (other buffer)
                            __syncwarp();
                            if (laneid_volatile() == 0) s_pdbl_col[t >> 5] = col + 1;
                            __syncwarp();
                        } else if (a.use_tma && k_lo == 0 && k == 7 && g_w0 + 32 <= a.tma_groups) {
                            tmem_wait_st();
                            tma_flush_half(tm_addr(), tma_buf(), &a.tmap, g_w0, col, 0, a.l2last);
                            if (blk + 1 < nblk) {  // defer the second half to the next block
                                if (laneid_volatile() == 0) {
                                    s_pend_col[t >> 5] = col + 1;
                                    s_pend_g[t >> 5] = g_w0;
                                }
                                __syncwarp();
                            } else {
                                tma_flush_half(tm_addr(), tma_buf(), &a.tmap, g_w0, col, 1, a.l2last);
                            }
                        } else if (k_lo == 0 && k == 7 && ((a.row_bytes | col) & 7) == 0 && a.row_bytes < (1ull << 32))
                            rowmajor_store_tmem_sectors(tm_addr() + dbl_off(B), s_row0 + (t & ~31u),
                                                        s_nvalid + (t & ~31u), a.row_bytes, col, a.l2last);
                        else
                            rowmajor_store_tmem(tm_addr() + dbl_off(B), s_row0[t], a.row_bytes, s_nvalid[t], k_lo, k,
                                                col);
                    }
                    else
                        rowmajor_store<SLOTS>(os_ptr(), s_row0[t], a.row_bytes, s_nvalid[t], k_lo, k, col);
                }
            }
        }

        // re-derive the item context (kept out of registers during the loop)
        item = *slot;
        lane = laneid_volatile();
        seg = item / a.units;
        w = item - seg * a.units;
        g = w * 32u + lane;
        const bool last = (seg + 1 == a.nseg);
        if (LAYOUT == L_CHECKSUM) {
            if (last) {
                uint64_t v = 0;
                if (g < a.G)
                    v = fmix64(uint64_t(acc & lane_mask(a, g)) ^ ((a.g_base + g) * 0x9E3779B97F4A7C15ull) ^
                               (a.t0 * 0xBF58476D1CE4E5B9ull));
#pragma unroll
                for (int off = 16; off > 0; off >>= 1) v += __shfl_xor_sync(0xFFFFFFFFu, v, off);
                if (lane == 0) atomicAdd(static_cast<unsigned long long*>(a.out), (unsigned long long)v);
            } else {
                __stcg(a.state + uint64_t(C::NSTATE) * a.Gp + g, acc);
            }
        }
        c.store(a.state, a.Gp, g);

        if (!a.persistent) break;
        if (!last) {
            __threadfence();
            __syncwarp();
            if (lane == 0) st_release(a.flags + w, uint32_t(seg + 1));
        }
        next_item(a, slot);
    }
    if constexpr (LAYOUT == L_ROW_MAJOR && TMEM) {
        if (a.use_tma && laneid_volatile() == 0) bulk_wait_all();  // smem boxes read, stores done
        __syncwarp();
        tmem_dealloc_cta(*reinterpret_cast<volatile uint32_t*>(&s_tmem), DBL || WIDE);
    }
}

}  // namespace bsk
