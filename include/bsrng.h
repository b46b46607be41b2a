/*
 * bsrng.h -- C ABI of the B200-native bitsliced keystream generator.
 *
 * The operation: many independent cipher instances (key, IV) each produce a
 * keystream; instances are laid out column-major ("bitsliced"), so one 32-bit
 * slice word holds the same-significance register bit of 32 instances
 * (sec. 4.1) and every register clock is straight-line
 * 32-lane logic (sec. 4.3; sec. 4.4 for
 * MICKEY 2.0: 200 slice words, 32 ciphers and 32 keystream bits per thread
 * per clock).  The paper's problem statement is "M pseudo-random bits from
 * many keyed generators", seeds partitioned across GPUs
 * (PAPER.md:781-789), each stream reproducible from its seed
 * (PAPER.md:799-803).
 *
 * Conventions
 *   - All functions are plain C; no CUDA or torch types appear.  `stream` is a
 *     cudaStream_t passed as void* (NULL = the legacy default stream).
 *   - A handle is bound to the CUDA device that was current at create time;
 *     every call switches to that device and restores the caller's device.
 *   - Integer-returning functions return BSRNG_OK (0) or a negative BSRNG_E*
 *     code; pointer-returning functions return NULL on failure.  In both cases
 *     bsrng_last_error() returns a thread-local, human-readable reason.
 *   - A handle is not thread-safe; distinct handles are independent.
 *     Multi-GPU use is one handle per device (one process per GPU).
 *   - There is no CPU fallback: without a usable sm_100 device, create fails
 *     with BSRNG_ECUDA.
 */
#ifndef BSRNG_H
#define BSRNG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    BSRNG_MICKEY2 = 1,     /* MICKEY 2.0, sec. 2.3.1, sec. 4.4   */
    BSRNG_GRAIN_V1 = 2,    /* Grain v1,   PAPER.md:339-357 sec. 2.3.3 (NEXT-1)   */
    BSRNG_AES128_CTR = 3,  /* AES-128-CTR, sec. 2.3.2 (NEXT-2)  */
    BSRNG_LFSR128 = 4      /* bitsliced LFSR of PAPER.md:545-596 sec. 4.3 (NEXT-4):
                              x^128+x^29+x^27+x^2+1, state = 16-byte key, no IV */
} bsrng_cipher;

/* Output layouts of bsrng_generate (sec. 4.5 leaves the
 * global output order unspecified; reading R9 defines these). */
typedef enum {
    /* instance i's bits at out + i*(bits/8) bytes.  MICKEY: first bit = MSB of
     * byte 0 (the specification's byte strings).  Grain: first bit = LSB.    */
    BSRNG_ROW_MAJOR = 0,
    /* uint32 out[bits][G]: bit j of word [t][g] = keystream bit t of instance
     * 32g+j (G = ceil(n/32)); padding lanes are 0.                           */
    BSRNG_SLICED = 1,
    /* one uint64: sum over groups g (mod 2^64) of
     *   fmix64(acc_g ^ (g_global * 0x9E3779B97F4A7C15) ^ (t0 * 0xBF58476D1CE4E5B9))
     * acc_g = XOR of this call's slice words of group g (padding lanes 0),
     * t0 = clocks generated before this call, g_global = first_instance/32 + g,
     * fmix64 = the SplitMix64 finaliser.  Additive, so it reduces exactly with
     * a uint64 sum across shards.                                             */
    BSRNG_CHECKSUM = 2
} bsrng_layout;

enum {
    BSRNG_OK = 0,
    BSRNG_EINVAL = -1,      /* bad argument (NULL, n == 0, bits % 32, layout, alignment,
                               iv_bits, a stream of another device)                      */
    BSRNG_ENOMEM = -2,      /* device / pinned-host allocation failed, or all 11 AES
                               round-key slots are taken (one per live AES handle)       */
    BSRNG_ECUDA = -3,       /* CUDA launch/runtime error (message in last_error)          */
    BSRNG_ERANGE = -4,      /* cumulative keystream bits per key/IV would exceed the
                               cipher's limit: MICKEY 2.0 2^40 (the spec's limit,
                               PAPER.md:254-256, reading R10); Grain v1, AES-128-CTR
                               and the LFSR 2^62 (the 64-bit bit counter)               */
    BSRNG_EUNSUPPORTED = -5 /* cipher/layout combination not built                        */
};

/* flags for bsrng_create_ex / bsrng_rekey */
enum {
    BSRNG_INPUT_HOST = 0,   /* keys/ivs are host pointers: copied into a handle-owned
                               pinned buffer during the call, then H2D stream-ordered;
                               the caller may reuse its buffers as soon as it returns  */
    BSRNG_INPUT_DEVICE = 1  /* keys/ivs are device pointers on the handle's device,
                               read by kernels on `stream`: they must stay unchanged
                               until the stream has passed the call                   */
};

typedef struct bsrng bsrng_t;

/*
 * bsrng_create -- allocate device state for n instances, slice their keys/IVs
 * and run the initialisation clocks (MICKEY: iv_bits + 80 + 100 CLOCK_KG with
 * mixing, spec [5]); synchronous on the legacy stream.
 *   keys: HOST, row-major uint8[n][key_bytes]   (MICKEY/Grain 10 B, LFSR 16 B;
 *         AES-128-CTR: ONE 16-byte key shared by all instances)
 *   ivs : HOST, row-major uint8[n][iv_bytes]    (MICKEY 10 B = 80-bit IV, the
 *         paper's benchmark IV; Grain 8 B; AES 16 B initial
 *         128-bit big-endian counter block; LFSR none: ivs may be NULL)
 *   n   : number of instances, >= 1 (padded internally to 32*ceil(n/32))
 * Ownership: inputs are copied; the caller keeps its buffers.
 */
bsrng_t* bsrng_create(bsrng_cipher cipher, const uint8_t* keys, const uint8_t* ivs, uint64_t n);

/*
 * bsrng_create_ex -- as bsrng_create, plus:
 *   iv_bits          : MICKEY IV length in bits, any value in 0..80 (the spec's
 *                      range; IV bit i = bit 7 - i%8 of byte
 *                      i/8; the IV row stride is still 10 B); Grain must be 64;
 *                      AES 128; LFSR 0.
 *   first_instance_id: global id of instance 0 (must be a multiple of 32); used
 *                      only to make CHECKSUM shard-invariant.
 *   flags            : BSRNG_INPUT_HOST or BSRNG_INPUT_DEVICE.
 *   stream           : work is enqueued on `stream` (which must belong to the
 *                      current device, else EINVAL); the call synchronises it
 *                      before returning.
 * AES-128-CTR handles each take one of 11 constant-memory round-key slots
 * (released by bsrng_destroy); a 12th live AES handle fails with ENOMEM.
 */
bsrng_t* bsrng_create_ex(bsrng_cipher cipher, const uint8_t* keys, const uint8_t* ivs,
                         uint32_t iv_bits, uint64_t n, uint64_t first_instance_id,
                         uint32_t flags, void* stream);

/*
 * bsrng_rekey -- re-initialise every instance of an existing handle with new
 * keys/IVs (same n, iv_bits): slice + initialisation clocks into the handle's
 * state, resetting its bit counter.  Asynchronous on `stream`: no host
 * synchronisation (AES: the key expansion runs on the device and its round
 * keys reach the handle's constant-memory slot by a stream-ordered copy).
 * Host inputs (BSRNG_INPUT_HOST) are copied into a handle-owned pinned buffer
 * before the call returns, so the caller may overwrite them immediately (the
 * call waits only for the previous rekey's copy out of that buffer).  Device
 * inputs (BSRNG_INPUT_DEVICE) must stay valid until `stream` passes the call.
 * Errors: EINVAL (NULL, unknown flags, a stream of another device), ENOMEM,
 * ECUDA.
 */
int bsrng_rekey(bsrng_t* h, const uint8_t* keys, const uint8_t* ivs, uint32_t flags,
                void* stream);

/*
 * bsrng_generate -- continue every instance's keystream by bits_per_instance
 * bits (stateful: consecutive calls concatenate) and write them to `out` in
 * `layout`.  Asynchronous on `stream`.
 *   out  : DEVICE memory, caller-owned, bsrng_out_bytes(h, bits, layout) bytes,
 *          16-byte aligned (CHECKSUM: 8-byte aligned; it is overwritten).
 *   bits_per_instance: multiple of 32 (AES: of 128); 0 is a no-op.  Calls of
 *          more than 2^31 bits per instance run as several time segments of
 *          one launch (the same result as one pass).
 *   stream: must belong to the handle's device (else EINVAL); NULL = the
 *          legacy default stream.  AES ROW_MAJOR calls of >= 4096 bits with a
 *          < 4096-bit remainder run that remainder on a handle-owned side
 *          stream forked from and joined back into `stream` by events, so
 *          the call stays ordered after earlier and before later work on
 *          `stream` (and is capturable in a CUDA graph).  Calls on one handle
 *          must not run concurrently on different streams.
 * Errors: EINVAL (NULL, alignment, bits, layout, stream), ERANGE (cumulative
 * bits per instance above the cipher's limit, see BSRNG_ERANGE), ECUDA.
 */
int bsrng_generate(bsrng_t* h, void* out, uint64_t bits_per_instance, bsrng_layout layout,
                   void* stream);

/*
 * bsrng_generate_host -- as bsrng_generate but `host_out` is HOST memory of
 * bsrng_out_bytes bytes (any alignment); the data is produced on the device in
 * chunks of at most 1 GiB (a handle-owned device bounce buffer) and copied
 * back; synchronises `stream` before returning.  CHECKSUM: 8 bytes.
 */
int bsrng_generate_host(bsrng_t* h, void* host_out, uint64_t bits_per_instance,
                        bsrng_layout layout, void* stream);

/* Bytes `out` must hold for one generate call (0 if h is NULL or args bad). */
uint64_t bsrng_out_bytes(const bsrng_t* h, uint64_t bits_per_instance, bsrng_layout layout);

/* Number of instances n, groups G = ceil(n/32), bits generated so far. */
uint64_t bsrng_num_instances(const bsrng_t* h);
uint64_t bsrng_num_groups(const bsrng_t* h);
uint64_t bsrng_bits_done(const bsrng_t* h);

/*
 * bsrng_copy_state -- copy the sliced cipher state to HOST memory (synchronous):
 * MICKEY: uint32[200][G] (rows 0..99 = R bits r_0..r_99, rows 100..199 = S
 * bits s_0..s_99); Grain v1: uint32[160][G] (rows 0..79 = LFSR s_0..s_79,
 * rows 80..159 = NFSR b_0..b_79).  Bit j of word [i][g] = that bit of
 * instance 32g+j.
 * `words` is the capacity of host_out in uint32 words.  Returns the number of
 * words written (>0) or a negative error code.
 */
int64_t bsrng_copy_state(const bsrng_t* h, uint32_t* host_out, uint64_t words);

/*
 * bsrng_set_option -- tuning knobs (for sweeps; defaults are the tuned ones).
 *   "sched"      : 0 = one thread per group for the whole call (calls of more
 *                  than 2^31 bits still use the queue), 1 = persistent,
 *                  time-segmented work queue (default)
 *   "seg_clocks" : clocks per work item when sched = 1 (multiple of 32; 0 = auto)
 *   "ctas_per_sm": resident CTAs per SM for the persistent grid (0 = auto)
 *   "unroll"     : clocks per loop iteration: Grain / LFSR 32 (default) or 16;
 *                  MICKEY 4 (the only one built); 0 = default
 *   "rm_ws"      : ROW_MAJOR kernel: -1 auto, 1 warp-specialised (a clock-loop
 *                  warp and a writer warp per SMSP; the writer transposes into
 *                  tensor memory and flushes 64 B per row; auto for MICKEY
 *                  and Grain when every warp-unit gets its own SMSP, unless
 *                  rm_tmem / rm_wide are set; AES: the block-lane kernel),
 *                  2 two writer warps per clock-loop warp (two streams per
 *                  SM, 128 B per row per flush, each writer two 32 B sectors
 *                  of it; LFSR only, its auto choice), 0 plain
 *   "rm_tmem"    : ROW_MAJOR plain kernel: stage the row segments in tensor
 *                  memory (TMEM, 256 columns per CTA, two CTAs per SM) (1)
 *                  or in shared memory (0); -1 = cipher default (MICKEY /
 *                  Grain 1, LFSR 0).  Setting it (or
 *                  rm_wide = 1) selects the plain kernel unless rm_ws is set
 *   "rm_tma"     : TMEM staging: whole-sector flushes of warps whose rows are
 *                  all real as TMA tensor stores when the row stride is a
 *                  multiple of 16 B (1, default) or as 8 B stores (0)
 *   "rm_dbl"     : TMEM staging with one CTA per SM and one time segment:
 *                  double-buffered staging (512 columns), the previous sector
 *                  period flushed 4 rows per block (1, default) or a single
 *                  buffer (0)
 *   "rm_wide"    : ROW_MAJOR plain kernel: 64 B TMEM staging per row with one
 *                  clock-loop warp per SMSP (1) or not (0, default)
 *   "rm_l2last"  : ROW_MAJOR 32 B flushes (TMA / 8 B stores) with an L2
 *                  evict_last hint (1, default) or evict-first (0)
 *   "rm_phase"   : writer-warp kernel (rm_ws = 1): stagger the warp-units'
 *                  64 B flush periods by 0, 2, .., 14 blocks (unit mod 8) so
 *                  that they do not all write at once (1), or flush every
 *                  unit in the same block (0); -1 (default) = on when the row
 *                  stride is not a multiple of 16 B (the paper's 552 B rows)
 *   "init_fused" : create/rekey: slicing fused into the initialisation kernel
 *                  (1, default) or the separate ballot slice (+ preclock)
 *                  kernels (0)
 * Returns BSRNG_OK or BSRNG_EINVAL for an unknown key/value.
 */
int bsrng_set_option(bsrng_t* h, const char* key, int64_t value);

/* Frees all device memory of the handle.  NULL-safe. */
void bsrng_destroy(bsrng_t* h);

/* Thread-local message for the last failure on this thread ("" if none). */
const char* bsrng_last_error(void);

/* Number of kernel launches this library has issued (process-wide counter). */
uint64_t bsrng_launch_count(void);

#ifdef __cplusplus
}
#endif

#endif /* BSRNG_H */
