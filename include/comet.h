/*
 * comet.h -- C ABI of libcomet.so, the B200 (sm_100a) W4Ax hot path of COMET
 * (Liu et al., "COMET: Towards Practical W4A4KV4 LLMs Serving", ASPLOS'25).
 * Citations "P:Lnnn" are lines of the paper text; DESIGN.md has the readings R*.
 *
 * The path ("O = WX"):   Y[M,N] = X[M,K] . W[N,K]^T
 *   1. comet_quantize_act : FMPQ -- every 128-channel block of every token row is quantised
 *      symmetric min-max to INT4 (qmax 7) or, for blocks tagged as outlier blocks, INT8
 *      (qmax 127), one FP32 scale per (token, block)  (R1-R5).
 *   2. comet_pack_weight  : INT4 weight codes [-8,7] -> packed nibbles (R14).
 *   3. comet_plan_create  : the SM scheduler -- a persistent-CTA work list over
 *      (output tile x K-block) units, either whole tiles balanced by cost (tile remapping,
 *      P:L220) or a stream-K split of tiles across CTAs (tile decomposition).
 *   4. comet_w4ax_gemm    : packed W4 x A4/A8 GEMM, exact integer per-block accumulation on
 *      the tcgen05 tensor cores, per-block dequantisation into FP32 and the s_w epilogue
 *      (P:L164-178).
 *
 * Conventions
 *   - Every pointer named *_dev / documented "device" is a CUDA device pointer owned by the
 *     caller; the library never frees caller memory.  *_host pointers are host memory read
 *     synchronously during the call.
 *   - Every launch is asynchronous on the given stream (cudaStream_t passed as void*; NULL =
 *     legacy default stream).  No call allocates or synchronises on the hot path
 *     (comet_quantize_act, comet_pack_weight, comet_w4ax_gemm).
 *   - Errors: every function returns a comet_status_t; nothing throws or aborts across the
 *     ABI.  Arguments are validated before any launch; on error nothing is launched.
 *     comet_last_error() returns a thread-local detail string for the last failure.
 *   - Shapes: K % 128 == 0 (FMPQ block k = 128); N % 128 == 0; M >= 1 (any value;
 *     ragged tails are handled); K <= 131072, N <= 1048576, M <= 2^31-1.
 *   - Alignment: every device pointer 16-byte aligned; ldx (elements) with ldx*2 % 16 == 0;
 *     ldy (elements) with ldy*sizeof(y) % 16 == 0 (ldy >= N).
 *   - Requires an sm_100a device (B200); otherwise COMET_ERR_NOT_SM100A.
 */
#ifndef COMET_H_
#define COMET_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define COMET_BLOCK_K 128   /* FMPQ block: k = 128 channels */
#define COMET_TILE_W  128   /* weight rows per output tile (MMA M) */
#define COMET_SCALE_PAD 16  /* token dimension of per-token arrays is padded to Mp = roundup(M,16) */

typedef enum {
  COMET_OK = 0,
  COMET_ERR_INVALID_ARG = 1,
  COMET_ERR_UNSUPPORTED_SHAPE = 2,
  COMET_ERR_MISALIGNED = 3,
  COMET_ERR_NOT_SM100A = 4,
  COMET_ERR_WORKSPACE_TOO_SMALL = 5,
  COMET_ERR_CUDA = 6
} comet_status_t;

typedef enum { COMET_F16 = 0, COMET_BF16 = 1, COMET_F32 = 2 } comet_dtype_t;

/* ------------------------------------------------------------------------------------------
 * Activation packed layout ("mixed-precision data layout", reading R15)
 *
 * For X[M,K] with nb = K/128 blocks and Mp = roundup(M, 16), the buffer `act_packed`
 * (comet_act_packed_bytes(M,K) bytes, 256-byte aligned) holds, at the byte offsets returned
 * by comet_act_layout():
 *
 *   codes [M][K]  uint8, row-major (row stride K bytes).  Byte (m,k), block b = k/128:
 *                   tags[b] == 0 (INT4 block): the E4M3 encoding of the INT4 code q in [-7,7]
 *                     (every integer |q| <= 7 is exact in E4M3:  0 -> 0x00, 1 -> 0x38,
 *                      2 -> 0x40, 3 -> 0x44, 4 -> 0x48, 5 -> 0x4A, 6 -> 0x4C, 7 -> 0x4E,
 *                      negative = 0x80 | encoding of |q|; -0 is never produced);
 *                   tags[b] == 1 (INT8 block): the two's-complement byte of q in [-127,127].
 *   qsum  [nb][Mp] int16:  qsum[b][m] = sum_{k in block b} q[m,k]   (exact; 0 for m >= M)
 *   corr  [Mp]     float:  corr[m] = 8 * sum_{b : tags[b]==0} scale[b][m] * qsum[b][m]
 *                          (binary32 sum, order implementation-defined; used by the GEMM to
 *                           undo the offset-binary weight encoding)
 *
 * act_scales [nb][Mp] float (separate buffer, 16-byte aligned):
 *   act_scales[b*Mp + m] = s_a[m,b] = amax / qmax (binary32), 0 for an all-zero block and
 *   for m >= M.
 * ---------------------------------------------------------------------------------------- */
typedef struct {
  size_t codes_off;     /* always 0 */
  size_t qsum_off;
  size_t corr_off;
  size_t total_bytes;
  int64_t Mp;           /* padded token count */
  int64_t nb;           /* K / 128 */
} comet_act_layout_t;

comet_status_t comet_act_layout(int64_t M, int64_t K, comet_act_layout_t* out);
size_t comet_act_packed_bytes(int64_t M, int64_t K);
/* number of floats of act_scales: nb * Mp */
size_t comet_act_scales_count(int64_t M, int64_t K);

/*
 * FMPQ activation quantisation.
 *   x          device, [M][ldx] float16 (xdt = COMET_F16) or bfloat16 (COMET_BF16), row-major.
 *   tags_host  host, [K/128] uint8, nonzero = INT8 (outlier) block.  Read synchronously.
 *   perm_dev   NULL (channels in input order) or device [K] int32: the runtime channel
 *              permutation of FMPQ (Fig. 4(d)) fused into the quantiser -- channel
 *              k of the quantised row is input channel perm_dev[k], x'[m,k] = x[m, perm[k]],
 *              and everything below (blocks, tags, codes, scales) refers to x'.  Must be a
 *              permutation of [0, K) (entries outside are clamped into range: defined but
 *              meaningless); the weights must be packed with the same permutation
 *              (comet_pack_weight_perm).  Requires K <= 32768 (the kernel stages whole rows
 *              and the permutation in shared memory), else COMET_ERR_UNSUPPORTED_SHAPE.
 *   act_packed device, comet_act_packed_bytes(M,K) bytes, written completely.
 *   act_scales device, comet_act_scales_count(M,K) floats, written completely.
 * Per (m, b): amax = max|x|; qmax = 127 if tags[b] else 7; amax == 0 -> s = 0 and codes 0;
 * else s = amax/qmax, r = qmax/amax (binary32, correctly rounded), q = clamp(rint(x*r))
 * with rint = round-half-even and x*r one binary32 product (NaN -> 0).  Inputs must be
 * finite.  Bit-exact with the CPU oracle.
 */
comet_status_t comet_quantize_act(const void* x, comet_dtype_t xdt, int64_t M, int64_t K,
                                  int64_t ldx, const uint8_t* tags_host, const int32_t* perm_dev,
                                  void* act_packed, float* act_scales, void* stream);

/* ------------------------------------------------------------------------------------------
 * Weight packed layout ("location switch" + "zero extension", reading R14)
 *
 * w_packed: N*K/2 bytes in 1 KB tiles of 16 rows x one 128-channel block, the tile of
 * (row tile n/16, block b) at byte ((n/16) * (K/128) + b) * 1024, inside it row n % 16 at
 * + (n % 16) * 64 (row-tiled: each 16-row group's K-blocks are contiguous, so a kernel that
 * walks K for a group of rows streams contiguous memory; N % 16 == 0).  Within a row's 64 B,
 * for every group of eight consecutive channels k = 8g .. 8g+7 (g relative to the block), the
 * little-endian 32-bit word at byte 4 (g % 16) has byte i (i = 0..3) equal to
 *        (u[8g+i] & 0xF) | (u[8g+i+4] << 4),      u = w + 8  (offset binary, 0..15).
 * Then (word & 0x0F0F0F0F) holds u[8g..8g+3] and ((word >> 4) & 0x0F0F0F0F) holds
 * u[8g+4..8g+7], one per byte, in channel order: widening costs 3 instructions per 8 values.
 * A byte 0x0u read as E4M3 is exactly u * 2^-9 (subnormal/first binade), so the widened
 * bytes feed the FP8 tensor core directly; (u << 4) ^ 0x80 is the int8 16*w for INT8 blocks.
 * The layout is opaque to callers beyond its size; comet_pack_weight(_perm) write it.
 * ---------------------------------------------------------------------------------------- */
size_t comet_weight_packed_bytes(int64_t N, int64_t K);
/* w_codes_dev: device [N][K] int8 codes in [-8,7] (values outside are masked to 4 bits). */
comet_status_t comet_pack_weight(const int8_t* w_codes_dev, int64_t N, int64_t K, void* w_packed,
                                 void* stream);
/* Offline weight side of the channel permutation ("the corresponding positions in the
 * weight matrix also need to be permuted"): packs W'[n,k] = W[n, perm_dev[k]] in the layout
 * above.  perm_dev: device [K] int32, a permutation of [0, K) (entries outside are clamped).
 * NULL perm_dev is the identity (same as comet_pack_weight). */
comet_status_t comet_pack_weight_perm(const int8_t* w_codes_dev, int64_t N, int64_t K,
                                      const int32_t* perm_dev, void* w_packed, void* stream);

/* ------------------------------------------------------------------------------------------
 * Offline calibration of the channel permutation and the precision tags ("we
 * utilize sampled activations from the calibration dataset to locate outlier channels and
 * apply permutation to group these channels into a single block"; reading R8/R16).
 * ---------------------------------------------------------------------------------------- */
/* amax_dev[k] = max_m |x[m,k]| over the calibration rows (device [K] float, written
 * completely; exact).  x as in comet_quantize_act (device, [M][ldx] f16 / bf16). */
comet_status_t comet_channel_amax(const void* x, comet_dtype_t xdt, int64_t M, int64_t K,
                                  int64_t ldx, float* amax_dev, void* stream);
/* Host, synchronous, no device needed.  amax_host: [K] per-channel max-abs (finite, >= 0).
 * med = median of amax_host in binary64 (mean of the two central values when K is even);
 * channel k is an outlier iff (double)amax_host[k] > ratio * med (ratio > 0; the paper's
 * "tenfold" is ratio = 10).  Writes perm_host[K] = the outlier channels in ascending
 * order followed by the other channels in ascending order, tags_host[K/128] = 1 for the first
 * ceil(n_outliers/128) blocks (the blocks that now hold outliers) and 0 for the rest, and
 * *n_outliers (may be NULL).  K % 128 == 0. */
comet_status_t comet_calibrate_perm(const float* amax_host, int64_t K, double ratio,
                                    int32_t* perm_host, uint8_t* tags_host, int64_t* n_outliers);

/* ------------------------------------------------------------------------------------------
 * KV4: INT4 KV-cache quantisation (the "KV4" of W4A4KV4; "a channel-wise 4-bit
 * quantization strategy for the KV cache", "channel-wise asymmetric INT4 group
 * quantization"; reading R17).  A K or V cache tensor kv[T][C] (T tokens, C = KV heads x
 * head_dim channels) is quantised per (group g of `group` consecutive tokens, channel c):
 *   mn = min x, mx = max x over the group's tokens; d = mx - mn (binary32);
 *   s = d / 15, r = 15 / d (correctly rounded; d == 0 -> s = r = 0);
 *   q = clamp(rint_half_even((x - mn) * r), 0, 15)     (binary32, never contracted)
 *   dequantised x_hat = mn + q * s (two binary32 roundings), rounded to f16/bf16.
 * Layouts (device, caller-owned):
 *   kv4_codes  [T][C/2] uint8: byte (t, j) = q[t][2j] | q[t][2j+1] << 4
 *   kv4_scales [ceil(T/group)][C] float = s;   kv4_mins [ceil(T/group)][C] float = mn
 * Constraints: T >= 1, C % 64 == 0, group in {32, 64, 128, 256}; ld (elements) >= C with
 * ld*2 % 16 == 0; pointers 16-byte aligned; inputs finite.  Bit-exact with the CPU oracle.
 * ---------------------------------------------------------------------------------------- */
comet_status_t comet_kv4_quantize(const void* kv, comet_dtype_t dt, int64_t T, int64_t C,
                                  int64_t ld, int group, uint8_t* kv4_codes, float* kv4_scales,
                                  float* kv4_mins, void* stream);
comet_status_t comet_kv4_dequantize(const uint8_t* kv4_codes, const float* kv4_scales,
                                    const float* kv4_mins, int64_t T, int64_t C, int group,
                                    void* out, comet_dtype_t odt, int64_t ldo, void* stream);

/* ------------------------------------------------------------------------------------------
 * Tile scheduler ("fine-grained SM scheduling")
 * ---------------------------------------------------------------------------------------- */
typedef struct comet_plan_s* comet_plan_t;   /* opaque, library-owned, immutable after create */

typedef struct {
  int tile_n;          /* orientation 1: tokens per output tile (MMA N): 16, 32, 64 or 128; 0 = auto */
  int num_sms;         /* persistent CTAs (one per SM); 0 = query the current device */
  int split_mode;      /* 0 = whole tiles onto the least-loaded CTA (no fix-up);
                          1 = tile decomposition: stream-K contiguous K-ranges;
                          2 = naive: (tile, K-block) units round-robin (Fig. 8b/c);
                          3 = unit remapping: units longest-first onto the least-loaded CTA
                              (Fig. 8d);
                         -1 = auto (stream-K when whole tiles fill < 92 % of the last wave) */
  float cost_int4;     /* planner cost of one INT4 K-block unit (default 1.0) */
  float cost_int8;     /* planner cost of one INT8 K-block unit (default 1.0 on B200) */
  int stages;          /* shared-memory ring depth: 0 = auto; any other value must equal the
                          depth the plan's kernel is compiled with (reported by
                          comet_plan_info().stages), else COMET_ERR_INVALID_ARG */
  int device_plan;     /* 1 (default) = upload the work list to the device at create time;
                          0 = host-only plan (comet_plan_describe only; CPU-safe) */
  int orientation;     /* 0 = auto (3 when M >= 256, 2 when M >= 128, 4 when M <= 8 and the
                              packed weights take >= 32 MiB, or >= 8 MiB with N >= K, else 1);
                          1 = weights on the MMA M side: tile = 128 weights x tile_n tokens
                              (decode-sized M; weights widened into TMEM);
                          2 = tokens on the MMA M side: tile = 128 tokens x tile_w weights
                              (prefill; weights widened into shared memory), tile_n ignored;
                          3 = as 2 on a tcgen05 CTA pair: tile = 256 tokens x tile_w weights,
                              each SM widens half the weights; num_ctas counts pairs;
                          4 = decode, M <= 8, warp-level tensor cores (mma.sync u8 x s8):
                              weights streamed by cp.async into per-warp rings, units
                              (128-weight group, K-block) cut into one contiguous range per
                              CTA, partials summed in CTA order by a second (dependent)
                              launch; per-channel s_w only, no debug outputs, needs the
                              plan's workspace; tile_n / tile_w / split_mode ignored */
  int tile_w;          /* orientations 2/3: weights per output tile (MMA N): 128, 160, 192, or
                          256 (orientation 3 only);
                          0 = auto (256 for orientation 3, 192 for 2).  Ignored for
                          orientation 1 (always 128). */
  int reserved[4];
} comet_sched_config;

/* Fill *cfg with the defaults (tile_n 0, num_sms 0, split_mode -1, costs 1/1, stages 0,
 * device_plan 1). */
void comet_sched_config_default(comet_sched_config* cfg);

/*
 * Build the work list for Y[M,N] = X[M,K] W[N,K]^T with the given block tags.
 *   tags_host  host [K/128] uint8 (copied into the plan).
 *   cfg        NULL = defaults.
 *   out        receives the plan.
 *   workspace_bytes  receives the device workspace comet_w4ax_gemm needs (stream-K partials
 *              and flags); may be 0.
 * Not on the hot path: may allocate device memory (the work list) when device_plan = 1.
 */
comet_status_t comet_plan_create(int64_t M, int64_t N, int64_t K, const uint8_t* tags_host,
                                 const comet_sched_config* cfg, comet_plan_t* out,
                                 size_t* workspace_bytes);
comet_status_t comet_plan_destroy(comet_plan_t plan);

typedef struct {
  int64_t M, N, K;
  int tile_n, num_ctas, split_mode, stages;
  int orientation, tile_w;  /* kernel orientation (1/2) and weights per output tile */
  int64_t n_tiles;         /* output tiles = ceil(N/tile_w) * ceil(M/tile_n) */
  int64_t n_items;         /* work items in the list */
  int64_t n_split_tiles;   /* tiles shared by more than one CTA */
  double max_cta_cost;     /* planner makespan (sum of unit costs on the busiest CTA) */
  double mean_cta_cost;
} comet_plan_info_t;
comet_status_t comet_plan_info(comet_plan_t plan, comet_plan_info_t* info);

/* Export the work list: items[4*i + {0,1,2,3}] = {cta, tile, kb_begin, kb_end} for the
 * i-th item (CTAs' items consecutive, in execution order).  *n_items = count written. */
comet_status_t comet_plan_describe(comet_plan_t plan, int32_t* items, int64_t max_items,
                                   int64_t* n_items);

/*
 * The W4Ax GEMM.   y[m, n] = s_w[n] * sum_b s_a[m,b] * acc_b[m,n]
 *   act_packed, act_scales  from comet_quantize_act with the plan's M, K and tags.
 *   w_packed                from comet_pack_weight (N*K/2 bytes, row-tiled, see above).
 *   w_scales                device [N] float (per-output-channel, reading R7).
 *   y                       device [M][ldy] of ydt (F16 / BF16 / F32), row-major.
 *   debug_acc               NULL, or device [M][N] int32: sum_b acc_b[m,n] in code units
 *                           (bit-exact integer accumulators; slower debug kernel).
 *   debug_acc_blocks        NULL, or device [K/128][M][N] int32 per-block acc_b (tiny shapes).
 *   workspace               device, >= the plan's workspace_bytes (may be NULL if 0).  Zero it
 *                           once before its first use: every completed launch leaves its
 *                           flag / counter words zero again, so it may then be reused by any
 *                           later call of any plan without clearing (flags also carry a
 *                           process-wide launch counter), but it must not be used by two GEMMs
 *                           in flight at the same time, and must be re-zeroed after a launch
 *                           that failed.
 * The persistent grid is sized at plan time to what the occupancy calculator admits as
 * co-resident (the stream-K owner of a split tile waits for the other units' partials); a
 * fix-up or pipeline wait that exceeds 4 s (only possible if another kernel holds the SMs that
 * long) traps, i.e. the launch fails with a CUDA error instead of hanging the device.
 */
comet_status_t comet_w4ax_gemm(comet_plan_t plan, const void* act_packed, const float* act_scales,
                               const void* w_packed, const float* w_scales, void* y,
                               comet_dtype_t ydt, int64_t ldy, int32_t* debug_acc,
                               int32_t* debug_acc_blocks, void* workspace, size_t ws_bytes,
                               void* stream);

/* The decode layer without a kernel-1 launch (kernel 1 fused into the GEMM, the
 * per-token quantisation of P:L126 / P:L136-138 as comet_quantize_act defines it):
 *   Y = W4Ax(FMPQ(x), W)      for M <= 8 and plans with orientation 4, or orientation 1 with
 *                              16-token tiles
 * x: device [M][ldx] F16 or BF16 (ldx >= K, x and ldx*2 16-byte aligned).  Orientation 1: each
 * pipeline stage's input rows arrive by TMA and one warp per CTA quantises them into the MMA's
 * operand slot (one launch).  Orientation 4: every CTA quantises the K-blocks of its range from
 * x into shared memory before its weight loop (the GEMM launch, plus the plan's reduction
 * launch).  Both use comet_quantize_act's arithmetic -- identical codes, scales and code sums --
 * so there is no activation buffer; the offset-binary weight term is removed per block (every
 * block sum is exact), so outputs equal the two-launch path's within FP32 reassociation, and bit
 * for bit when every partial sum is exact.  Other arguments as comet_w4ax_gemm; other plans get
 * COMET_ERR_UNSUPPORTED_SHAPE.  Launched as a programmatic dependent of the preceding kernel on
 * the stream (its weight stream starts while that kernel finishes; x is read only after it
 * completed). */
comet_status_t comet_w4ax_linear(comet_plan_t plan, const void* x, comet_dtype_t xdt, int64_t ldx,
                                 const void* w_packed, const float* w_scales, void* y,
                                 comet_dtype_t ydt, int64_t ldy, void* workspace, size_t ws_bytes,
                                 void* stream);

/* NEXT-3: group-wise weight scales (the "group size of 128" weight scaling of the paper's QoQ
 * comparison; reading R18): one scale per (128-channel block b, output channel n),
 *   Y[m,n] = sum_b s_a[m,b] * s_w[b,n] * acc_b[m,n]          (acc_b = sum_{k in b} q w, exact)
 * w_scales_grouped: device [K/128][N] float (block-major).  Arguments otherwise as
 * comet_w4ax_gemm (no per-block debug output).  Runs on the weights-on-MMA-M kernel (plan
 * orientation 1, the default for M < 128) or on the 256-wide prefill pair kernel (orientation 3,
 * tile_w 256, the default for M >= 256; no debug accumulators there); other plans get
 * COMET_ERR_UNSUPPORTED_SHAPE. */
comet_status_t comet_w4ax_gemm_grouped(comet_plan_t plan, const void* act_packed, const float* act_scales,
                                       const void* w_packed, const float* w_scales_grouped, void* y,
                                       comet_dtype_t ydt, int64_t ldy, int32_t* debug_acc,
                                       void* workspace, size_t ws_bytes, void* stream);


/* ------------------------------------------------------------------------------------------
 * NEXT-2: the row-parallel layer's reduction fused into the GEMM epilogue (the
 * paper lists "operator pipelining" as future work).  Under tensor parallelism a
 * row-parallel layer (e.g. LLaMA down, K sharded over `world` ranks at 128-channel block
 * boundaries, each rank quantising its own K shard) produces per-rank FP32 partials
 * Y_r = X_r W_r^T that must be summed.  Instead of writing Y_r and running an all-reduce, the
 * prefill pair kernel's epilogue stores every finished tile row m straight into the receive
 * buffer of the rank that owns row m (owner = m / ms, ms = ceil(M / world)) -- peer memory
 * over NVLink, so the transfer of one tile overlaps the MMAs of the next -- and the owner sums
 * the `world` slots in rank order (deterministic): a reduce-scatter over token rows.
 *
 *   recv buffer of every rank: device [world][ms][N] float (comet_rs_recv_bytes bytes),
 *     slot [src][m - owner * ms][n] = Y_src[m][n]; recv_bufs_host[i] = rank i's buffer as
 *     mapped in this process (peer pointers, e.g. from torch symmetric memory).
 *   comet_w4ax_gemm_rs  this rank's GEMM (plan orientation 3, else COMET_ERR_UNSUPPORTED_SHAPE;
 *     arguments as comet_w4ax_gemm); writes its slot in every owner's buffer.
 *   comet_rs_reduce     on the owner, after EVERY rank's comet_w4ax_gemm_rs has completed (the
 *     caller orders them, e.g. a barrier across ranks): y[i][n] = sum_src recv[src][i][n] for
 *     this rank's rows i < min(ms, M - rank * ms) (output rows rank * ms + i), into y [rows][ldy]
 *     of ydt.  world in 1..8.
 * ---------------------------------------------------------------------------------------- */
size_t comet_rs_recv_bytes(int64_t M, int64_t N, int world);
comet_status_t comet_w4ax_gemm_rs(comet_plan_t plan, const void* act_packed, const float* act_scales,
                                  const void* w_packed, const float* w_scales, float* const* recv_bufs_host,
                                  int world, int rank, void* workspace, size_t ws_bytes, void* stream);
comet_status_t comet_rs_reduce(const float* recv_local, int world, int rank, int64_t M, int64_t N, void* y,
                               comet_dtype_t ydt, int64_t ldy, void* stream);

/*
 * Convenience: the whole hot path for one linear layer with HOST buffers (used for the
 * end-to-end measurement).  Copies x_host [M][K] (F16/BF16, pinned host memory for overlap) to
 * the device, quantises, runs the GEMM and copies y [M][N] back to y_host.
 *   M < 2048: all on `stream`, in order.
 *   M >= 2048: pipelined over chunks of 1024 token rows -- chunk c's H2D copy (an internal copy
 *   stream), its quantise + GEMM (on `stream`, with an internal sub-plan of the same scheduler
 *   configuration) and its D2H copy (a second internal copy stream) overlap the neighbouring
 *   chunks' transfers and compute.  The uploads start at once (ordered only after the previous
 *   call with this plan has finished reading its scratch); quantise + GEMM follow the work
 *   already queued on `stream`; the downloads run on the internal stream.
 * comet_w4ax_linear_host returns when y_host is complete.  The _async form returns at once:
 * x_host and y_host must stay valid, and y_host is complete after comet_linear_host_wait(plan)
 * (or a device synchronize); for M < 2048 completion of `stream` suffices.  Device scratch (x,
 * act, scales, y, the sub-plans' fix-up workspace) comes from `scratch` (256-byte aligned, at
 * least comet_linear_scratch_bytes(plan, xdt, ydt) bytes; that call also builds the sub-plans)
 * and must not be used by anything else while calls are in flight.  `workspace` is the plan's
 * own fix-up workspace (used when M < 2048).  Not thread-safe per plan.
 */
size_t comet_linear_scratch_bytes(comet_plan_t plan, comet_dtype_t xdt, comet_dtype_t ydt);
comet_status_t comet_w4ax_linear_host(comet_plan_t plan, const void* x_host, comet_dtype_t xdt,
                                      const void* w_packed, const float* w_scales, void* y_host,
                                      comet_dtype_t ydt, void* scratch, size_t scratch_bytes,
                                      void* workspace, size_t ws_bytes, void* stream);
comet_status_t comet_w4ax_linear_host_async(comet_plan_t plan, const void* x_host, comet_dtype_t xdt,
                                            const void* w_packed, const float* w_scales, void* y_host,
                                            comet_dtype_t ydt, void* scratch, size_t scratch_bytes,
                                            void* workspace, size_t ws_bytes, void* stream);
/* Block until the downloads of the last comet_w4ax_linear_host(_async) call with `plan` are done. */
comet_status_t comet_linear_host_wait(comet_plan_t plan);

/* ------------------------------------------------------------------------------------------
 * Diagnostic: the GEMM kernels' widening step on caller-chosen packed words (P:L202-206
 * "location switch" + "zero extension"; layout R14 above), for the exhaustive widening pin.
 * For i in [0, n): word v = (first_word + i) mod 2^32, eight consecutive channels packed as
 * above; out_dev[2i] = bytes u[0..3], out_dev[2i+1] = bytes u[4..7] (u = nibble value 0..15,
 * i.e. the E4M3 operand u * 2^-9 of an INT4 block); with int8_block != 0 each byte is instead
 * the s8 value 16 * (u - 8) of an INT8 block.  out_dev: device [n][2] uint32, 8-byte aligned.
 * n in [0, 2^32].  Asynchronous on `stream`.
 * ---------------------------------------------------------------------------------------- */
comet_status_t comet_debug_widen(uint64_t first_word, int64_t n, int int8_block, uint32_t* out_dev,
                                 void* stream);

const char* comet_status_string(comet_status_t s);
const char* comet_last_error(void);
/* Library version string and the number of kernels the last comet_w4ax_gemm /
 * comet_quantize_act call launched (for launch accounting). */
const char* comet_version(void);
int comet_last_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* COMET_H_ */
