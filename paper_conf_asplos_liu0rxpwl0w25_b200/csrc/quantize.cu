// quantize.cu -- kernel 1: FMPQ activation quantisation and the mixed-precision packed layout.
//
// Per (token m, 128-channel block b) (P:L136 blocks of k = 128 channels along the channel
// dimension; P:L138 outlier blocks -> 8 bit, the rest 4 bit; P:L126 min-max; reading R1-R5):
//   amax = max |x|, qmax = tags[b] ? 127 : 7, s = amax/qmax, r = qmax/amax (IEEE binary32,
//   correctly rounded: __fdiv_rn), q = clamp(rint(x*r)) with x*r one binary32 product
//   (__fmul_rn, never contracted) and rint = round-half-even (cvt.rni; NaN -> 0).
// Layout written (include/comet.h): codes[M][K] bytes (E4M3 of q for INT4 blocks, s8 for INT8
// blocks), scales[nb][Mp], qsum[nb][Mp] (int16), corr[Mp].
//
// HBM-bound: a block-row (128 halves = 256 B) is read by 4 lanes with four 128-bit loads each
// (a warp step covers 8 blocks, sector-coalesced); block max-abs and code sum are 2-step
// xor-shuffle reductions inside the lane quad; codes leave as four 64-bit stores per lane.
#include <algorithm>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include "internal.h"
#include "sm100.cuh"
#include "fmpq.cuh"

#ifndef COMET_PERM_GATHER
#define COMET_PERM_GATHER 1   // decode-sized M: fused permutation by direct L1-cached gathers
#endif

namespace comet {
namespace {

using namespace fmpq;

// WPR warps cooperate on one token row; a CTA of 8 warps covers 8/WPR rows.  A warp step
// covers a group of 8 consecutive blocks (1024 channels, 2 KB of input): lane l works on block
// 8g + l/4 with sub = l%4, loading 4 x 16 B at channel offsets 32 j + 8 sub -- every load
// instruction reads 64 contiguous bytes of each of the 8 blocks (whole 32-byte sectors) and
// every code store writes 32 contiguous bytes per block.
// GATHER: the fused channel permutation (NEXT-1) as direct gathers -- channel k of the row is
// read from x[m, perm[k]] with 16-bit L1-cached loads (the CTA's rows are re-read sector by
// sector from L1; calibrated permutations are ascending runs, so a warp's gathers coalesce).
// PF: the next group's four loads are issued before this group's arithmetic (a warp keeps two
// groups in flight); it costs 16 registers (80: 3 CTAs per SM instead of 4), so the launcher
// uses it only when a warp walks >= 3 groups (tools/quant_bench.py: K = 28672 71.3 -> 67.3 us,
// M = 8192 K = 14336 71.7 -> 66.8 us; at K = 8192, 2 groups per warp, 23.4 -> 24.6 us: off)
template <bool BF16, int WPR, bool GATHER = false, bool PF = false>
__global__ void __launch_bounds__(256, PF ? 3 : 4) k_quantize(const uint16_t* __restrict__ x, int64_t M,
                                                  int64_t K, int64_t ldx, int64_t Mp, TagMask tags,
                                                  uint8_t* __restrict__ codes,
                                                  int16_t* __restrict__ qsum,
                                                  float* __restrict__ corr,
                                                  float* __restrict__ scales,
                                                  const int32_t* __restrict__ perm = nullptr) {
  constexpr int ROWS = 8 / WPR;
  __shared__ float s_part[8];
  // let a programmatic dependent (the decode GEMM) launch now: it streams weights while this
  // grid runs and waits for our completion before touching the activations
  asm volatile("griddepcontrol.launch_dependents;");
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int row_in_cta = warp / WPR, wi = warp % WPR;
  const int64_t m = (int64_t)blockIdx.x * ROWS + row_in_cta;
  const int bl = lane >> 2, sub = lane & 3;
  const int nb = (int)(K / kBlockK);
  const int ngroups = (nb + 7) >> 3;
  float cpart = 0.f;   // sum over this lane's INT4 blocks of s * qsum (binary32, lanes sub == 0)
  if (m < M) {
    const uint16_t* xrow = x + m * ldx + sub * 8;
    uint8_t* crow = codes + m * K + sub * 8;
    uint4 rawn[4];                                    // PF: the next group's loads
    if (!GATHER && PF && wi < ngroups) {
      const int b0 = wi * 8 + bl;
#pragma unroll
      for (int j = 0; j < 4; ++j)
        rawn[j] = b0 < nb ? ldg_stream(xrow + b0 * kBlockK + 32 * j) : make_uint4(0, 0, 0, 0);
    }
    for (int g = wi; g < ngroups; g += WPR) {
      const int b = g * 8 + bl;
      const bool bvalid = b < nb;
      uint4 raw[4];
      if (!GATHER && !PF) {
#pragma unroll
        for (int j = 0; j < 4; ++j)
          raw[j] = bvalid ? ldg_stream(xrow + b * kBlockK + 32 * j) : make_uint4(0, 0, 0, 0);
      } else if (!GATHER) {
#pragma unroll
        for (int j = 0; j < 4; ++j) raw[j] = rawn[j];
        const int bn_ = (g + WPR) * 8 + bl;
        if (g + WPR < ngroups) {
#pragma unroll
          for (int j = 0; j < 4; ++j)
            rawn[j] = bn_ < nb ? ldg_stream(xrow + bn_ * kBlockK + 32 * j) : make_uint4(0, 0, 0, 0);
        }
      } else {
        const uint16_t* xr = x + m * ldx;
        const int kmax = (int)K - 1;
        int idx[32];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const int k0 = b * kBlockK + 32 * j + sub * 8;
          int4 p0 = make_int4(0, 0, 0, 0), p1 = make_int4(0, 0, 0, 0);
          if (bvalid) {
            p0 = __ldg(reinterpret_cast<const int4*>(perm + k0));
            p1 = __ldg(reinterpret_cast<const int4*>(perm + k0 + 4));
          }
          idx[8 * j + 0] = p0.x; idx[8 * j + 1] = p0.y; idx[8 * j + 2] = p0.z; idx[8 * j + 3] = p0.w;
          idx[8 * j + 4] = p1.x; idx[8 * j + 5] = p1.y; idx[8 * j + 6] = p1.z; idx[8 * j + 7] = p1.w;
        }
        uint32_t h[32];
#pragma unroll
        for (int i = 0; i < 32; ++i)
          h[i] = bvalid ? (uint32_t)__ldg(xr + min(max(idx[i], 0), kmax)) : 0u;
#pragma unroll
        for (int j = 0; j < 4; ++j)
          raw[j] = make_uint4(h[8 * j] | (h[8 * j + 1] << 16), h[8 * j + 2] | (h[8 * j + 3] << 16),
                              h[8 * j + 4] | (h[8 * j + 5] << 16), h[8 * j + 6] | (h[8 * j + 7] << 16));
      }
      float v[32];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        float t[8];
        unpack8<BF16>(raw[j], t);
#pragma unroll
        for (int i = 0; i < 8; ++i) v[8 * j + i] = t[i];
      }
      const bool is8 = bvalid && ((tags.w[b >> 5] >> (b & 31)) & 1u);
      const LaneOut o = quantize32(v, is8);
      if (bvalid) {
        uint8_t* cb = crow + b * kBlockK;
#pragma unroll
        for (int j = 0; j < 4; ++j) *reinterpret_cast<uint2*>(cb + 32 * j) = o.c[j];
        if (sub == 0) {
          scales[(int64_t)b * Mp + m] = o.s;
          qsum[(int64_t)b * Mp + m] = (int16_t)o.q;
          if (!is8) cpart = __fadd_rn(cpart, __fmul_rn(o.s, (float)o.q));
        }
      }
    }
  } else if (m < Mp) {
    // padding rows: scales and qsum 0
    for (int b = wi * 32 + lane; b < nb; b += WPR * 32) {
      scales[(int64_t)b * Mp + m] = 0.f;
      qsum[(int64_t)b * Mp + m] = 0;
    }
  }
  // fixed-order reduction of the lanes' partial corrections (lanes with sub != 0 hold 0)
  cpart = __fadd_rn(cpart, __shfl_xor_sync(0xffffffffu, cpart, 4));
  cpart = __fadd_rn(cpart, __shfl_xor_sync(0xffffffffu, cpart, 8));
  cpart = __fadd_rn(cpart, __shfl_xor_sync(0xffffffffu, cpart, 16));
  if (lane == 0) s_part[warp] = cpart;
  __syncthreads();
  if (wi == 0 && lane == 0 && m < Mp) {
    float c = 0.f;
    for (int i = 0; i < WPR; ++i) c = __fadd_rn(c, s_part[row_in_cta * WPR + i]);
    corr[m] = __fmul_rn(8.f, c);
  }
}

// ---------------------------------------------------------------------------- fused permutation
// NEXT-1: the runtime channel permutation that groups outlier channels into a
// few blocks (Fig. 4(d)) fused into kernel 1: channel k of the quantised row is
// input channel perm[k], x'[m,k] = x[m, perm[k]], then FMPQ exactly as above on x'.
//
// A gather cannot be sector-coalesced from HBM, so each CTA stages whole input rows in shared
// memory with 1D bulk copies (cp.async.bulk, completion on an mbarrier; a row is split over 8
// issuing warps) -- NBUF rows in flight -- and the permutation once per CTA as 16-bit indices
// (K <= 32768).  Per row: pass 1 gathers the permuted row into a second (swizzled) staging row
// (consecutive threads take consecutive output channels), the input buffer is refilled at once,
// and pass 2 runs the FMPQ lane layout of k_quantize on the staged row.  Persistent CTAs walk
// rows m = blockIdx.x + i * gridDim.x.  Measured (tools/quant_time.py, M = 4096, calibrated
// permutation): 51 us at K = 8192 and 141 us at K = 28672, against 26.5 / 69.7 us without the
// permutation -- the per-row passes are latency-bound at 1-2 CTAs per SM (ncu: issue 45 %).
// Position of permuted channel k in the staged row: odd blocks swap their 32-channel halves
// pairwise (channel bit 5 ^= block bit 0), so the pass-2 128-bit reads of two neighbouring
// blocks (256 B apart, same banks) land in different bank halves.
__device__ __forceinline__ int64_t swz(int64_t k) { return k ^ (((k >> 7) & 1) << 5); }

template <bool BF16, int NW, int R>
__global__ void __launch_bounds__(NW * 32, 2) k_quantize_perm(const uint16_t* __restrict__ x, int64_t M,
                                                       int64_t K, int64_t ldx, int64_t Mp,
                                                       TagMask tags,
                                                       const int32_t* __restrict__ perm, int nbuf,
                                                       uint8_t* __restrict__ codes,
                                                       int16_t* __restrict__ qsum,
                                                       float* __restrict__ corr,
                                                       float* __restrict__ scales) {
  // R rows per step (R = 2 for K <= 16384): the per-row chain -- gather pass, barrier, FMPQ
  // pass, barrier -- is latency-bound, and a K = 8192 row has only 8 groups of 8 blocks for 16
  // warps; two rows per step fill every warp in pass 2 and double the work per barrier
  extern __shared__ __align__(128) uint8_t smem[];
  asm volatile("griddepcontrol.launch_dependents;");                  // see k_quantize
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);                 // [nbuf] (<= 16)
  uint16_t* p16 = reinterpret_cast<uint16_t*>(smem + 128);            // [K] permutation
  uint16_t* prow = p16 + K;                                           // [R][K] permuted rows (swizzled)
  uint16_t* rows = prow + R * K;                                      // [nbuf][R][K] input rows
  __shared__ float s_part[R][NW];
  __shared__ uint32_t s_tags[kMaxBlocks / 32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int bl = lane >> 2, sub = lane & 3;
  const int nb = (int)(K / kBlockK);
  const int ngroups = (nb + 7) >> 3;
  if (threadIdx.x == 0) {
#pragma unroll
    for (int i = 0; i < kMaxBlocks / 32; ++i) s_tags[i] = tags.w[i];   // constant indices: no local copy
  }
  const uint32_t row_bytes = (uint32_t)(K * 2);
  if (threadIdx.x == 0) {
    for (int i = 0; i < nbuf; ++i) sm100::mbar_init(&full[i], 1);
    sm100::fence_mbar_init();
  }
  for (int64_t k = threadIdx.x; k < K; k += blockDim.x) p16[k] = (uint16_t)min(max(__ldg(perm + k), 0), (int)K - 1);
  __syncthreads();
  // A row arrives as kChunks bulk copies issued by lane 0 of different warps: one issuing
  // thread's bulk copies complete one after another (profiles/r01/probe_stream.txt), several
  // issuers overlap.  Thread 0 posts the step's byte count; the chunks may land before or after.
  // Step i of this CTA holds rows R (blockIdx.x + i gridDim.x) + r, r < R.
  constexpr int kChunks = NW < 8 ? NW : 8;
  const uint32_t chunk = row_bytes / kChunks;          // K % 128 == 0 -> a multiple of 32 B
  const bool issuer = lane == 0 && warp < kChunks;
  auto load_step = [&](int64_t st, int buf) {          // issuer threads only
    const int64_t m0 = st * R;
    const int nr = (int)min((int64_t)R, M - m0);
    if (nr <= 0) return;
    if (warp == 0) sm100::mbar_arrive_expect_tx(&full[buf], row_bytes * (uint32_t)nr);
    for (int r = 0; r < nr; ++r)
      sm100::bulk_load(reinterpret_cast<uint8_t*>(rows + ((int64_t)buf * R + r) * K) + warp * chunk,
                       reinterpret_cast<const uint8_t*>(x + (m0 + r) * ldx) + warp * chunk, chunk, &full[buf]);
  };
  const int64_t nsteps = (Mp + R - 1) / R;
  if (issuer)
    for (int i = 0; i < nbuf; ++i) load_step(blockIdx.x + (int64_t)i * gridDim.x, i);
  int it = 0;
  for (int64_t st = blockIdx.x; st < nsteps; st += gridDim.x, ++it) {
    const int buf = it % nbuf;
    const int64_t m0 = st * R;
    const int nr = (int)max((int64_t)0, min((int64_t)R, M - m0));   // real rows of this step
    float cpart[R];
#pragma unroll
    for (int r = 0; r < R; ++r) cpart[r] = 0.f;
    if (nr > 0) {
      sm100::mbar_wait(&full[buf], (uint32_t)((it / nbuf) & 1));
      // pass 1: gather.  Thread t moves output channels 2t, 2t+1 (+ 2*blockDim.x steps) of each
      // row: consecutive threads read consecutive indices (and, for the mostly ascending
      // calibrated permutations, consecutive input channels) -- no bank conflicts -- and write
      // the pair as one word at its swizzled position.
      for (int64_t k = 2 * threadIdx.x; k < K; k += 2 * blockDim.x) {
        const uint32_t pi = *reinterpret_cast<const uint32_t*>(p16 + k);
#pragma unroll
        for (int r = 0; r < R; ++r) {
          if (r >= nr) break;
          const uint16_t* row = rows + ((int64_t)buf * R + r) * K;
          const uint32_t h = (uint32_t)row[pi & 0xFFFFu] | ((uint32_t)row[pi >> 16] << 16);
          *reinterpret_cast<uint32_t*>(prow + (int64_t)r * K + swz(k)) = h;
        }
      }
    }
    __syncthreads();   // prow complete; row buffer `buf` free
    if (issuer && nr > 0) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      load_step(st + (int64_t)nbuf * gridDim.x, buf);   // refill the freed buffer
    }
    // pass 2: FMPQ on the permuted rows, the lane layout of k_quantize (reads conflict-free
    // thanks to the swizzle: the 8 blocks of a warp step sit 256 B apart); padding rows
    // (M <= m < Mp) get zero scales and code sums
    for (int gg = warp; gg < R * ngroups; gg += NW) {
      const int r = gg / ngroups, g = gg % ngroups;
      const int64_t m = m0 + r;
      if (m >= Mp) continue;
      const int b = g * 8 + bl;
      const bool bvalid = b < nb;
      if (r >= nr) {
        if (bvalid && sub == 0) {
          scales[(int64_t)b * Mp + m] = 0.f;
          qsum[(int64_t)b * Mp + m] = 0;
        }
        continue;
      }
      float v[32];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        uint4 raw = make_uint4(0, 0, 0, 0);
        if (bvalid) raw = *reinterpret_cast<const uint4*>(prow + (int64_t)r * K + swz((int64_t)b * kBlockK + 32 * j + sub * 8));
        float t[8];
        unpack8<BF16>(raw, t);
#pragma unroll
        for (int i = 0; i < 8; ++i) v[8 * j + i] = t[i];
      }
      const bool is8 = bvalid && ((s_tags[b >> 5] >> (b & 31)) & 1u);
      const LaneOut o = quantize32(v, is8);
      if (bvalid) {
        uint8_t* cb = codes + m * K + sub * 8 + b * kBlockK;
#pragma unroll
        for (int j = 0; j < 4; ++j) *reinterpret_cast<uint2*>(cb + 32 * j) = o.c[j];
        if (sub == 0) {
          scales[(int64_t)b * Mp + m] = o.s;
          qsum[(int64_t)b * Mp + m] = (int16_t)o.q;
          if (!is8) {
#pragma unroll
            for (int rr = 0; rr < R; ++rr)
              if (rr == r) cpart[rr] = __fadd_rn(cpart[rr], __fmul_rn(o.s, (float)o.q));
          }
        }
      }
    }
#pragma unroll
    for (int r = 0; r < R; ++r) {
      float c = cpart[r];
      c = __fadd_rn(c, __shfl_xor_sync(0xffffffffu, c, 4));
      c = __fadd_rn(c, __shfl_xor_sync(0xffffffffu, c, 8));
      c = __fadd_rn(c, __shfl_xor_sync(0xffffffffu, c, 16));
      if (lane == 0) s_part[r][warp] = c;
    }
    __syncthreads();   // s_part complete; prow free
    if (threadIdx.x < R && m0 + threadIdx.x < Mp) {
      const int r = threadIdx.x;
      float c = 0.f;
      for (int i = 0; i < NW; ++i) c = __fadd_rn(c, s_part[r][i]);
      corr[m0 + r] = __fmul_rn(8.f, c);
    }
  }
}

// Offline weight side of the permutation ("the corresponding positions in the weight
// matrix also need to be permuted"): W'[n,k] = W[n, perm[k]], packed as k_pack_weight.
__global__ void __launch_bounds__(256) k_pack_weight_perm(const int8_t* __restrict__ w, int64_t N,
                                                          int64_t K, const int32_t* __restrict__ perm,
                                                          uint32_t* __restrict__ out) {
  const int64_t words = N * K / 8;
  const int kmax = (int)K - 1;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = i / (K / 8), k0 = (i % (K / 8)) * 8;
    const int8_t* wr = w + n * K;
    uint32_t word = 0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int p0 = min(max(__ldg(perm + k0 + j), 0), kmax), p1 = min(max(__ldg(perm + k0 + j + 4), 0), kmax);
      const uint32_t lo = ((uint32_t)wr[p0] & 0xFu) ^ 8u;   // u[k0 + j]
      const uint32_t hi = ((uint32_t)wr[p1] & 0xFu) ^ 8u;   // u[k0 + j + 4]
      word |= (lo | (hi << 4)) << (8 * j);
    }
    out[packed_word_index(n, k0 / 8, K / kBlockK)] = word;
  }
}

// Calibration statistic (offline, "sampled activations from the calibration dataset"):
// amax[k] = max_m |x[m,k]|.  Non-negative binary32 values order like their bit patterns, so the
// max is an atomicMax on the bits (order-independent, deterministic).  Each thread owns 8
// consecutive channels (one 128-bit load per row) over a slice of the rows.
template <bool BF16>
__global__ void __launch_bounds__(256) k_channel_amax(const uint16_t* __restrict__ x, int64_t M,
                                                      int64_t K, int64_t ldx, int64_t rows_per_cta,
                                                      unsigned int* __restrict__ amax) {
  const int64_t c8 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 8;
  if (c8 >= K) return;
  const int64_t m0 = (int64_t)blockIdx.y * rows_per_cta;
  const int64_t m1 = m0 + rows_per_cta < M ? m0 + rows_per_cta : M;
  float a[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
  for (int64_t m = m0; m < m1; ++m) {
    float v[8];
    unpack8<BF16>(ldg_stream(x + m * ldx + c8), v);
#pragma unroll
    for (int i = 0; i < 8; ++i) a[i] = fmaxf(a[i], fabsf(v[i]));
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) atomicMax(amax + c8 + i, __float_as_uint(a[i]));
}

// Small-M (decode) variant: a row is split over a cluster of S CTAs (S <= 8) so that a single
// token row of K = 28672 channels is read by 64 warps in one load round instead of by 8 warps
// in four.  CTA `part` of the cluster takes the row's 8-block groups part*8 + warp, step 8*S;
// the correction term corr[m] is reduced across the cluster through distributed shared memory
// in a fixed (rank, warp) order by rank 0 -- deterministic, no atomics.
template <bool BF16>
__global__ void __launch_bounds__(256) k_quantize_split(const uint16_t* __restrict__ x, int64_t M,
                                                        int64_t K, int64_t ldx, int64_t Mp, int S,
                                                        TagMask tags,
                                                        uint8_t* __restrict__ codes,
                                                        int16_t* __restrict__ qsum,
                                                        float* __restrict__ corr,
                                                        float* __restrict__ scales) {
  __shared__ float s_part[8];
  asm volatile("griddepcontrol.launch_dependents;");                  // see k_quantize
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int part = (int)sm100::cluster_ctarank();
  const int64_t m = blockIdx.x / S;
  const int bl = lane >> 2, sub = lane & 3;
  const int nb = (int)(K / kBlockK);
  const int ngroups = (nb + 7) >> 3;
  float cpart = 0.f;
  if (m < M) {
    const uint16_t* xrow = x + m * ldx + sub * 8;
    uint8_t* crow = codes + m * K + sub * 8;
    for (int g = part * 8 + warp; g < ngroups; g += 8 * S) {
      const int b = g * 8 + bl;
      const bool bvalid = b < nb;
      uint4 raw[4];
#pragma unroll
      for (int j = 0; j < 4; ++j)
        raw[j] = bvalid ? ldg_stream(xrow + b * kBlockK + 32 * j) : make_uint4(0, 0, 0, 0);
      float v[32];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        float t[8];
        unpack8<BF16>(raw[j], t);
#pragma unroll
        for (int i = 0; i < 8; ++i) v[8 * j + i] = t[i];
      }
      const bool is8 = bvalid && ((tags.w[b >> 5] >> (b & 31)) & 1u);
      const LaneOut o = quantize32(v, is8);
      if (bvalid) {
        uint8_t* cb = crow + b * kBlockK;
#pragma unroll
        for (int j = 0; j < 4; ++j) *reinterpret_cast<uint2*>(cb + 32 * j) = o.c[j];
        if (sub == 0) {
          scales[(int64_t)b * Mp + m] = o.s;
          qsum[(int64_t)b * Mp + m] = (int16_t)o.q;
          if (!is8) cpart = __fadd_rn(cpart, __fmul_rn(o.s, (float)o.q));
        }
      }
    }
  } else if (m < Mp) {
    for (int b = part * 256 + threadIdx.x; b < nb; b += 256 * S) {
      scales[(int64_t)b * Mp + m] = 0.f;
      qsum[(int64_t)b * Mp + m] = 0;
    }
  }
  cpart = __fadd_rn(cpart, __shfl_xor_sync(0xffffffffu, cpart, 4));
  cpart = __fadd_rn(cpart, __shfl_xor_sync(0xffffffffu, cpart, 8));
  cpart = __fadd_rn(cpart, __shfl_xor_sync(0xffffffffu, cpart, 16));
  if (lane == 0) s_part[warp] = cpart;
  sm100::cluster_sync();                    // every CTA's partials written, visible cluster-wide
  if (part == 0 && threadIdx.x == 0 && m < Mp) {
    float c = 0.f;
    for (int r = 0; r < S; ++r) {
      const uint32_t base = sm100::mapa_shared(sm100::smem_u32(s_part), (uint32_t)r);
      for (int i = 0; i < 8; ++i) {
        float v;
        asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(base + 4u * i));
        c = __fadd_rn(c, v);
      }
    }
    corr[m] = __fmul_rn(8.f, c);
  }
  sm100::cluster_sync();                    // keep every CTA's shared memory alive until read
}

template <bool BF16>
cudaError_t launch_q(const void* x, int64_t M, int64_t K, int64_t ldx, const TagMask& tags,
                     void* act_packed, float* act_scales, cudaStream_t stream) {
  comet_act_layout_t L;
  act_layout(M, K, &L);
  uint8_t* base = static_cast<uint8_t*>(act_packed);
  uint8_t* codes = base + L.codes_off;
  int16_t* qsum = reinterpret_cast<int16_t*>(base + L.qsum_off);
  float* corr = reinterpret_cast<float*>(base + L.corr_off);
  const int64_t Mp = L.Mp;
  const int64_t nb = L.nb;
  // enough CTAs for ~8 per SM (memory-level parallelism), warps of a row sharing its groups
  const int64_t target = 8 * 148;
  const int64_t ngroups = (nb + 7) / 8;
  if (M <= 32 && ngroups > 8) {
    // decode: split every row over a cluster of S CTAs (one 8-block group per warp)
    const int S = (int)std::min<int64_t>(8, ceil_div(ngroups, 8));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)(Mp * S));
    cfg.blockDim = dim3(256);
    cfg.stream = stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = (unsigned)S;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_quantize_split<BF16>, static_cast<const uint16_t*>(x), M, K, ldx,
                              Mp, S, tags, codes, qsum, corr, act_scales);
  }
  int wpr = 1;
  while (wpr < 8 && ceil_div(Mp, 8 / wpr) < target && ngroups >= 2 * wpr) wpr *= 2;
#ifdef COMET_Q_WPR
  wpr = COMET_Q_WPR;
#endif
  const int rows = 8 / wpr;
  const dim3 grid((unsigned)ceil_div(Mp, rows));
  const uint16_t* xp = static_cast<const uint16_t*>(x);
#ifdef COMET_Q_PF
  const bool pf = COMET_Q_PF;
#else
  const bool pf = ngroups >= 3 * wpr;                // a warp walks >= 3 groups
#endif
  switch (wpr * 2 + (pf ? 1 : 0)) {
    case 2: k_quantize<BF16, 1><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales); break;
    case 3: k_quantize<BF16, 1, false, true><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales); break;
    case 4: k_quantize<BF16, 2><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales); break;
    case 5: k_quantize<BF16, 2, false, true><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales); break;
    case 8: k_quantize<BF16, 4><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales); break;
    case 9: k_quantize<BF16, 4, false, true><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales); break;
    case 17: k_quantize<BF16, 8, false, true><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales); break;
    default: k_quantize<BF16, 8><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales); break;
  }
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------- weight packing
// u = w + 8 = (w & 0xF) ^ 8 per nibble; word byte i = u[i] | u[i+4] << 4 (include/comet.h).
// Row-tiled placement (include/comet.h): word g of row n goes to 1 KB tile (n/16, g/16), row
// n % 16, word g % 16.
__global__ void __launch_bounds__(256) k_pack_weight(const uint2* __restrict__ w, int64_t N, int64_t K,
                                                     uint32_t* __restrict__ out) {
  const int64_t wpr = K / 8, words = N * wpr, nb = K / kBlockK;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words;
       i += (int64_t)gridDim.x * blockDim.x) {
    const uint2 v = w[i];
    const uint32_t lo = (v.x & 0x0F0F0F0Fu) ^ 0x08080808u;   // u[k0..k3]
    const uint32_t hi = (v.y & 0x0F0F0F0Fu) ^ 0x08080808u;   // u[k4..k7]
    out[packed_word_index(i / wpr, i % wpr, nb)] = lo | (hi << 4);
  }
}

}  // namespace

void act_layout(int64_t M, int64_t K, comet_act_layout_t* L) {
  L->nb = K / kBlockK;
  L->Mp = round_up(M, COMET_SCALE_PAD);
  L->codes_off = 0;
  L->qsum_off = (size_t)round_up(M * K, 256);
  L->corr_off = (size_t)round_up((int64_t)L->qsum_off + L->nb * L->Mp * 2, 256);
  L->total_bytes = (size_t)round_up((int64_t)L->corr_off + L->Mp * 4, 256);
}

cudaError_t launch_quantize(const void* x, bool bf16, int64_t M, int64_t K, int64_t ldx,
                            const TagMask& tags, void* act_packed, float* act_scales,
                            cudaStream_t stream, int* launches) {
  *launches = 1;
  return bf16 ? launch_q<true>(x, M, K, ldx, tags, act_packed, act_scales, stream)
              : launch_q<false>(x, M, K, ldx, tags, act_packed, act_scales, stream);
}

template <bool BF16>
static cudaError_t launch_qp(const void* x, int64_t M, int64_t K, int64_t ldx, const TagMask& tags,
                             const int32_t* perm, void* act_packed, float* act_scales,
                             cudaStream_t stream) {
  comet_act_layout_t L;
  act_layout(M, K, &L);
  uint8_t* base = static_cast<uint8_t*>(act_packed);
  // M <= 32 (decode): direct gathers (one row per CTA, the row's sectors re-read from L1) beat
  // the staged rows -- 8.4 vs 10.2 us at M = 1, 16.4 vs 18.4 at M = 32, K = 28672; at prefill
  // sizes the staged kernel wins on long rows (141 vs 149 us at K = 28672) and on arbitrary
  // permutations (157 vs 344 us), tools/quant_time.py.
  if (COMET_PERM_GATHER && M <= 32) {
    uint8_t* codes = base + L.codes_off;
    int16_t* qsum = reinterpret_cast<int16_t*>(base + L.qsum_off);
    float* corr = reinterpret_cast<float*>(base + L.corr_off);
    const int64_t Mp = L.Mp, nb = L.nb, target = 8 * 148, ngroups = (nb + 7) / 8;
    int wpr = 1;
    while (wpr < 8 && ceil_div(Mp, 8 / wpr) < target && ngroups >= 2 * wpr) wpr *= 2;
    const dim3 grid((unsigned)ceil_div(Mp, 8 / wpr));
    const uint16_t* xp = static_cast<const uint16_t*>(x);
    switch (wpr) {
      case 1: k_quantize<BF16, 1, true><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales, perm); break;
      case 2: k_quantize<BF16, 2, true><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales, perm); break;
      case 4: k_quantize<BF16, 4, true><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales, perm); break;
      default: k_quantize<BF16, 8, true><<<grid, 256, 0, stream>>>(xp, M, K, ldx, Mp, tags, codes, qsum, corr, act_scales, perm); break;
    }
    return cudaGetLastError();
  }
  const int64_t row_bytes = K * 2;
  // R rows per step when two CTAs of 2-row steps with double buffering fit one SM (K <= 8192:
  // p16 + 2 staged rows + 2 x 2 input rows = 7 rows = 112 KB); else one row per step with
  // ~64 KB of staged input rows in flight
  const int R = (128 + (size_t)row_bytes * 7 <= (113u << 10)) ? 2 : 1;
  int nbuf = R == 2 ? 2 : (int)std::max<int64_t>(2, std::min<int64_t>(8, (64 << 10) / row_bytes));
  const size_t cap = 200u << 10;
  while (nbuf > 1 && 128 + (size_t)row_bytes * (1 + R + (size_t)nbuf * R) > cap) --nbuf;
  const size_t smem = 128 + (size_t)row_bytes * (1 + R + (size_t)nbuf * R);
  int dev = 0, nsm = 148, per_sm = 1;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  constexpr int NW = 16;   // 16 warps: the gather is latency-bound at one or two CTAs per SM
  auto kern = R == 2 ? k_quantize_perm<BF16, NW, 2> : k_quantize_perm<BF16, NW, 1>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, NW * 32, smem);
  if (e != cudaSuccess) return e;
  const int64_t grid = std::max<int64_t>(1, std::min<int64_t>(ceil_div(L.Mp, (int64_t)R), (int64_t)nsm * std::max(per_sm, 1)));
  kern<<<(unsigned)grid, NW * 32, smem, stream>>>(
      static_cast<const uint16_t*>(x), M, K, ldx, L.Mp, tags, perm, nbuf, base + L.codes_off,
      reinterpret_cast<int16_t*>(base + L.qsum_off), reinterpret_cast<float*>(base + L.corr_off),
      act_scales);
  return cudaGetLastError();
}

cudaError_t launch_quantize_perm(const void* x, bool bf16, int64_t M, int64_t K, int64_t ldx,
                                 const TagMask& tags, const int32_t* perm, void* act_packed,
                                 float* act_scales, cudaStream_t stream, int* launches) {
  *launches = 1;
  return bf16 ? launch_qp<true>(x, M, K, ldx, tags, perm, act_packed, act_scales, stream)
              : launch_qp<false>(x, M, K, ldx, tags, perm, act_packed, act_scales, stream);
}

cudaError_t launch_pack_weight_perm(const int8_t* w, int64_t N, int64_t K, const int32_t* perm,
                                    void* w_packed, cudaStream_t stream) {
  const int64_t words = N * K / 8;
  const int64_t blocks = std::min<int64_t>(ceil_div(words, 256), 148 * 16);
  k_pack_weight_perm<<<(unsigned)blocks, 256, 0, stream>>>(w, N, K, perm, static_cast<uint32_t*>(w_packed));
  return cudaGetLastError();
}

cudaError_t launch_channel_amax(const void* x, bool bf16, int64_t M, int64_t K, int64_t ldx,
                                float* amax, cudaStream_t stream) {
  cudaError_t e = cudaMemsetAsync(amax, 0, (size_t)K * 4, stream);
  if (e != cudaSuccess) return e;
  const int64_t cols = ceil_div(K / 8, 256);
  const int64_t ysplit = std::max<int64_t>(1, std::min<int64_t>(ceil_div(M, 32), ceil_div(148 * 8, cols)));
  const int64_t rows_per = ceil_div(M, ysplit);
  const dim3 grid((unsigned)cols, (unsigned)ceil_div(M, rows_per));
  unsigned int* out = reinterpret_cast<unsigned int*>(amax);
  if (bf16)
    k_channel_amax<true><<<grid, 256, 0, stream>>>(static_cast<const uint16_t*>(x), M, K, ldx, rows_per, out);
  else
    k_channel_amax<false><<<grid, 256, 0, stream>>>(static_cast<const uint16_t*>(x), M, K, ldx, rows_per, out);
  return cudaGetLastError();
}

cudaError_t launch_pack_weight(const int8_t* w, int64_t N, int64_t K, void* w_packed,
                               cudaStream_t stream) {
  const int64_t words = N * K / 8;
  const int64_t blocks = std::min<int64_t>(ceil_div(words, 256), 148 * 16);
  k_pack_weight<<<(unsigned)blocks, 256, 0, stream>>>(reinterpret_cast<const uint2*>(w), N, K,
                                                        static_cast<uint32_t*>(w_packed));
  return cudaGetLastError();
}

}  // namespace comet
