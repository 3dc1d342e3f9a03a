// gemm_v.cu -- the decode-regime W4Ax GEMM (plan orientation 4, M <= 8): weights streamed by
// cp.async into per-warp shared-memory rings, the product on the warp-level tensor-core path
// (mma.sync m16n8k32), partials of shared row groups summed by a dependent reduction launch.
//
//   Y[m, n] = s_w[n] * sum_b s_a[m,b] * acc_b[m,n],  acc_b = sum_{k in b} w[n,k] q[m,k]
//
//
// Why a second decode kernel.  At M <= 8 the layer is a weight stream (N x K/2 bytes against
// M x K codes): HBM-bound, with ~1 MAC per weight byte per token.  The tcgen05 decode kernel
// (gemm.cu, orientation 1) stages weights through TMA rings, widens them into TMEM and pays a
// barrier protocol per stage; its skeleton alone streams below the copy rate.
// Here every warp is its own weight pipeline: each lane cp.asyncs 16 B of row g and of row
// g + 8 per K-block (its warp's 16 rows = one 1 KB tile of the row-tiled layout, contiguous
// along K) into an S-deep ring it alone reads back -- no barrier in the loop -- widens in
// registers (3 instructions per 8 nibbles) and feeds 4 mma.sync per K-block.
//
// Work split (CTA-level stream-K): units = (group of 128 weight rows, K-block),
// group-major, cut into one contiguous range per CTA, equal to within one unit; warp w of the
// CTA takes rows 16 w .. 16 w + 15 of the group in every unit, so the CTA's 8 warps walk the
// same K-blocks and share one shared-memory copy of the activation codes of its range (staged
// once in the prologue as s8: from kernel 1's output, or -- FQ, comet_w4ax_linear -- quantised
// from x right there with kernel 1's arithmetic).  Each CTA stores one FP32 partial per group it
// touches ([128 rows][8 tokens] workspace slots); k_gemv_reduce -- a programmatic dependent
// launch, one CTA per group -- sums each group's partials in CTA order (deterministic), applies
// s_w and converts.
//
// Product per K-block (128 channels), one path for both block kinds: A = the weight nibbles
// u = w + 8 zero-extended to u8, B = the activation codes as s8 (INT8 blocks as stored, INT4
// blocks converted from their E4M3 bytes at staging); mma.sync m16n8k32 .s32.u8.s8 gives
// sum u q exactly, acc_b = d - 8 qsum[b][m] (exact), and the promotion adds s_a[m,b] acc_b in
// FP32 (reading R7 order: per block, then s_w once).
// K order inside a K-block: mma c (c = 0..3) of lane (g, t) takes packed word 4t + c of rows
// g and g + 8 (low nibbles -> A k-slots 4t.., high nibbles -> 16 + 4t..) and code bytes
// 32t + 8c .. + 7 of token g -- the same channel <-> slot map on both operands, so each lane
// loads 16 contiguous bytes of each of its two rows and 32 contiguous code bytes per K-block.
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include "internal.h"
#include "fmpq.cuh"

#ifndef COMET_GEMV_S
#define COMET_GEMV_S 8      // deepest ring (K-blocks in flight per warp, 1 KB stages); gemv_pick may take 6 or 4
#endif
#ifndef COMET_GEMV_CPS
#define COMET_GEMV_CPS 3    // CTAs (8 warps each) per SM, at most (shared memory decides, gemv_pick)
#endif

namespace comet {
namespace gemv {

constexpr int kRowsCta = 128;          // weight rows per CTA unit (8 warps x 16)
constexpr int kMaxStageBlocks = 128;   // activation blocks a CTA can stage (M = 8: 128 KB)

namespace {

struct VParams {
  const uint8_t* w;        // packed weights, row-tiled 1 KB tiles (include/comet.h)
  const uint8_t* codes;    // activation codes [M][K]
  const float* scales;     // s_a [nb][Mp]
  const int16_t* qsum;     // code sums [nb][Mp]
  float* part;             // partials [ctas][maxseg][128][8]
  const float* w_scales;   // s_w [N]
  const uint16_t* x;       // FQ: the layer input [M][ldx] f16 / bf16 (kernel 1 fused into the staging)
  int64_t ldx;
  int xbf16;
  void* y;
  int64_t M, N, K, Mp, ldy, units;
  int nb, maxseg, ctas, nbr, ydt;
  int early;               // trigger the dependent reduction launch at kernel start (small layers)
  TagMask tags;
};

__device__ __forceinline__ uint4 ldg_stream(const void* p) {   // weights: read once
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

__device__ __forceinline__ void mma_u8s8(int (&d)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3,
                                         uint32_t b0, uint32_t b1) {
  asm volatile("mma.sync.aligned.m16n8k32.row.col.s32.u8.s8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
               : "+r"(d[0]), "+r"(d[1]), "+r"(d[2]), "+r"(d[3])
               : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// s8 bytes of four E4M3 codes of integers |q| <= 7: E4M3 -> f16 (exact), + 1536 puts q in the
// low byte of the f16 pattern (0x6600 + q: ulp 1 on [1024, 2048)), a byte permute packs them.
__device__ __forceinline__ uint32_t e4m3x4_to_s8(uint32_t e) {
  uint32_t h0, h1;
  asm("{\n\t.reg .b16 lo, hi;\n\tmov.b32 {lo, hi}, %2;\n\t"
      "cvt.rn.f16x2.e4m3x2 %0, lo;\n\tcvt.rn.f16x2.e4m3x2 %1, hi;\n\t}\n"
      : "=r"(h0), "=r"(h1) : "r"(e), "r"(e));
  const uint32_t bias = 0x66006600u;   // f16x2 {1536, 1536}: 1536 + q in [1024, 2048), ulp 1
  asm("add.rn.f16x2 %0, %0, %1;" : "+r"(h0) : "r"(bias));
  asm("add.rn.f16x2 %0, %0, %1;" : "+r"(h1) : "r"(bias));
  return __byte_perm(h0, h1, 0x6420);
}

template <int S, bool FQ>
__global__ void __launch_bounds__(256, COMET_GEMV_CPS) k_gemv(const __grid_constant__ VParams P) {
  extern __shared__ __align__(16) uint8_t smem[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int M = (int)P.M;
  uint8_t* s_w = smem;                                                 // [8 warps][S][16 rows][64 B]
  uint8_t* s_x = smem + 8 * S * 1024;                                  // [nbr][M tokens][128 B] s8, swizzled
  float* s_s = reinterpret_cast<float*>(s_x + P.nbr * M * 128);        // [nbr][8] s_a
  int* s_q = reinterpret_cast<int*>(s_s + P.nbr * 8);                  // [nbr][4] qsum pairs
  const int cta = blockIdx.x;
  const int64_t u0 = P.units * cta / P.ctas, u1 = P.units * (cta + 1) / P.ctas;
  const int nb = P.nb;
  const int kb_s = (int)(u0 % nb);                                     // staging slot j <-> block (kb_s + j) % nb
  const int n_units = (int)(u1 - u0);
  // Weights: each lane copies 16 B of row g and of row g + 8 per unit into the warp's ring
  // (cp.async, no registers held) and reads back exactly those bytes, so a lane's own
  // cp.async.wait_group orders them -- no barrier.  Rows are 64 B apart in a stage: a phase of
  // eight lanes reads 128 contiguous bytes.
  const uint32_t ring = (uint32_t)__cvta_generic_to_shared(s_w + warp * S * 1024) + g * 64 + t * 16;
  // rows 16 warp .. of a group are one row tile of the packed layout: tile (grp * 8 + warp, b)
  // at ((grp * 8 + warp) * nb + b) KB -- each warp streams its tile row contiguously along K
  const uint8_t* wbase = P.w + (int64_t)warp * nb * 1024 + g * 64 + t * 16;   // + grp * 8 nb KB + b KB
  const int64_t grp_stride = (int64_t)8 * nb * 1024;
  int64_t lgrp = u0 / nb;
  int lb = (int)(u0 - lgrp * nb);
  int lslot = 0;
  auto issue = [&]() {                       // unit (lgrp, lb) -> ring slot lslot, advance
    const uint8_t* r0 = wbase + lgrp * grp_stride + lb * 1024;
    const uint32_t d = ring + lslot * 1024;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(r0) : "memory");
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d + 512), "l"(r0 + 512) : "memory");
    if (++lb == nb) { lb = 0; ++lgrp; }
    if (++lslot == S) lslot = 0;
  };
  // small layers: let the reduction launch now (its CTAs wait resident for this grid): qkv (42 MB)
  // 12.4 -> 11.6 us; on the 117 MB layers it costs 0.7 us (its CTAs take SM slots the GEMV's
  // last CTAs need), so they trigger after their weight loop
  if (P.early) asm volatile("griddepcontrol.launch_dependents;");
  // the weights are not written by the predecessor (kernel 1): stream them before the wait
  for (int k = 0; k < S - 1; ++k) {
    if (k < n_units) issue();
    asm volatile("cp.async.commit_group;" ::: "memory");
  }
  asm volatile("griddepcontrol.wait;" ::: "memory");
  // ---- stage the range's activation codes (s8), scales and code sums
  if constexpr (FQ) {
    // kernel 1 fused (comet_w4ax_linear): each lane quad quantises one (K-block, token) of the
    // range from x with kernel 1's own arithmetic (fmpq.cuh: the same codes, scales and code
    // sums bit for bit); INT4 codes go to shared memory as s8.  Tokens >= M keep s_a = qsum = 0.
    for (int i = threadIdx.x; i < P.nbr * 8; i += blockDim.x) {
      s_s[i] = 0.f;
      if ((i & 1) == 0) s_q[i >> 1] = 0;
    }
    __syncthreads();
    const int quad = threadIdx.x >> 2, sub = threadIdx.x & 3;
    const int npairs = P.nbr * M;
    for (int base = 0; base < npairs; base += 64) {              // warp-uniform trip count
      const int pr = base + quad;
      const bool ok = pr < npairs;
      const int j = ok ? pr / M : 0, m = ok ? pr - j * M : 0;
      const int kb = (kb_s + j) % nb;
      float v[32];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint4 raw = make_uint4(0, 0, 0, 0);
        if (ok) raw = __ldg(reinterpret_cast<const uint4*>(P.x + m * P.ldx + kb * 128 + 32 * q + 8 * sub));
        float tq[8];
        if (P.xbf16) fmpq::unpack8<true>(raw, tq); else fmpq::unpack8<false>(raw, tq);
#pragma unroll
        for (int e = 0; e < 8; ++e) v[8 * q + e] = tq[e];
      }
      const bool is8 = ok && ((P.tags.w[kb >> 5] >> (kb & 31)) & 1u);
      const fmpq::LaneOut o = fmpq::quantize32(v, is8);
      if (ok) {
        uint8_t* row = s_x + (j * M + m) * 128;
#pragma unroll
        for (int q = 0; q < 4; ++q) {            // channels 32q + 8 sub .. + 7: chunk 2q + sub/2, half sub&1
          uint2 c = o.c[q];
          if (!is8) { c.x = e4m3x4_to_s8(c.x); c.y = e4m3x4_to_s8(c.y); }
          *reinterpret_cast<uint2*>(row + (((2 * q + (sub >> 1)) ^ (m & 1)) << 4) + (sub & 1) * 8) = c;
        }
        if (sub == 0) {
          s_s[j * 8 + m] = o.s;
          reinterpret_cast<int16_t*>(s_q)[j * 8 + m] = (int16_t)o.q;
        }
      }
    }
  } else {
  for (int i = threadIdx.x; i < P.nbr * M * 8; i += blockDim.x) {   // 16-byte chunks
    const int j = i / (M * 8), r = i - j * (M * 8), m = r >> 3, ch = r & 7;
    const int kb = (kb_s + j) % nb;
    uint4 v = __ldg(reinterpret_cast<const uint4*>(P.codes + m * P.K + kb * 128 + ch * 16));
    if (!((P.tags.w[kb >> 5] >> (kb & 31)) & 1u)) {
      v.x = e4m3x4_to_s8(v.x); v.y = e4m3x4_to_s8(v.y); v.z = e4m3x4_to_s8(v.z); v.w = e4m3x4_to_s8(v.w);
    }
    // chunk ch of token m at chunk position ch ^ (m & 1): the reads of tokens g, g + 1 in one
    // phase of a 16-byte load land in different bank halves
    *reinterpret_cast<uint4*>(s_x + (j * M + m) * 128 + ((ch ^ (m & 1)) << 4)) = v;
  }
  for (int i = threadIdx.x; i < P.nbr * 8; i += blockDim.x) {
    const int j = i >> 3, m = i & 7;
    const int kb = (kb_s + j) % nb;
    s_s[i] = P.scales[(int64_t)kb * P.Mp + m];                       // rows >= M: 0 (kernel 1)
    if ((m & 1) == 0) s_q[i >> 1] = *reinterpret_cast<const int*>(P.qsum + (int64_t)kb * P.Mp + m);
  }
  }
  __syncthreads();

  float y[4] = {0.f, 0.f, 0.f, 0.f};         // (row g | g+8) x (token 2t | 2t+1)
  int seg = 0;
  auto flush = [&]() {
    float* dst = P.part + ((int64_t)(cta * P.maxseg + seg) * kRowsCta + warp * 16) * 8;
    *reinterpret_cast<float2*>(dst + g * 8 + 2 * t) = make_float2(y[0], y[1]);
    *reinterpret_cast<float2*>(dst + (g + 8) * 8 + 2 * t) = make_float2(y[2], y[3]);
  };
  const bool tok = g < M;                     // this lane's B-fragment token is real
  const uint32_t xa_off = g * 128 + (((2 * t) ^ (g & 1)) << 4), xb_off = g * 128 + (((2 * t + 1) ^ (g & 1)) << 4);
  int j = 0;                                  // staging slot of the unit being consumed
  int cb = kb_s;                              // its K-block
  int cslot = 0;                              // its ring slot
  for (int i = 0; i < n_units; ++i) {
    if (i + S - 1 < n_units) issue();         // unit i + S - 1 into the slot unit i - 1 left
    asm volatile("cp.async.commit_group;" ::: "memory");
    asm volatile("cp.async.wait_group %0;" ::"n"(S - 1) : "memory");   // unit i has landed
    if (cb == nb) {                           // a new row group (CTA-uniform)
      cb = 0;
      flush();
      ++seg;
      y[0] = y[1] = y[2] = y[3] = 0.f;
    }
    uint4 wa, wb;
    const uint32_t rs = ring + cslot * 1024;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(wa.x), "=r"(wa.y), "=r"(wa.z), "=r"(wa.w) : "r"(rs));
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(wb.x), "=r"(wb.y), "=r"(wb.z), "=r"(wb.w) : "r"(rs + 512));
    if (++cslot == S) cslot = 0;
    uint4 xa = make_uint4(0, 0, 0, 0), xb = make_uint4(0, 0, 0, 0);
    if (tok) {
      const uint8_t* xs = s_x + j * M * 128;
      xa = *reinterpret_cast<const uint4*>(xs + xa_off);
      xb = *reinterpret_cast<const uint4*>(xs + xb_off);
    }
    const float2 s = *reinterpret_cast<const float2*>(s_s + j * 8 + 2 * t);
    const int q2 = s_q[j * 4 + t];
    if (++j == P.nbr) j = 0;
    ++cb;
    const uint32_t wA[4] = {wa.x, wa.y, wa.z, wa.w}, wB[4] = {wb.x, wb.y, wb.z, wb.w};
    const uint32_t x[8] = {xa.x, xa.y, xa.z, xa.w, xb.x, xb.y, xb.z, xb.w};
    // two independent accumulation chains (K slices 0, 2 and 1, 3)
    int d0[4] = {0, 0, 0, 0}, d1[4] = {0, 0, 0, 0};
#pragma unroll
    for (int c = 0; c < 4; c += 2) {
      mma_u8s8(d0, wA[c] & 0x0F0F0F0Fu, wB[c] & 0x0F0F0F0Fu, (wA[c] >> 4) & 0x0F0F0F0Fu,
               (wB[c] >> 4) & 0x0F0F0F0Fu, x[2 * c], x[2 * c + 1]);
      mma_u8s8(d1, wA[c + 1] & 0x0F0F0F0Fu, wB[c + 1] & 0x0F0F0F0Fu, (wA[c + 1] >> 4) & 0x0F0F0F0Fu,
               (wB[c + 1] >> 4) & 0x0F0F0F0Fu, x[2 * c + 2], x[2 * c + 3]);
    }
    const int q0 = (int)(int16_t)(q2 & 0xFFFF), q1 = q2 >> 16;
    y[0] = __fmaf_rn(s.x, (float)(d0[0] + d1[0] - 8 * q0), y[0]);
    y[1] = __fmaf_rn(s.y, (float)(d0[1] + d1[1] - 8 * q1), y[1]);
    y[2] = __fmaf_rn(s.x, (float)(d0[2] + d1[2] - 8 * q0), y[2]);
    y[3] = __fmaf_rn(s.y, (float)(d0[3] + d1[3] - 8 * q1), y[3]);
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  // the reduction kernel may launch now; it waits for this grid's completion before reading
  if (!P.early) asm volatile("griddepcontrol.launch_dependents;");
  if (n_units > 0) flush();
}

// y[m][n] = s_w[n] * sum over the CTAs covering n's row group (in CTA order) of their partials.
// One CTA per row group, one thread per row: the group's contributing CTAs and their slots are
// computed once (the 64-bit divisions off the per-output path), then each thread reads its row's
// [8 tokens] from every slot with two 16-byte loads, all issued before the in-order sum.
constexpr int kMaxRed = 64;   // contributing CTAs a group can have (plan: at most one CTA per unit)
__global__ void __launch_bounds__(kRowsCta) k_gemv_reduce(const __grid_constant__ VParams P) {
  asm volatile("griddepcontrol.launch_dependents;");           // the next layer may start
  __shared__ int s_slot[kMaxRed];
  __shared__ int s_n;
  const int64_t grp = blockIdx.x;
  const int r = threadIdx.x;
  if (r == 0) {
    // CTA owning unit u: the largest c with floor(units c / ctas) <= u
    auto owner = [&](int64_t u) { return (int)(((u + 1) * P.ctas - 1) / P.units); };
    s_n = owner(grp * P.nb + P.nb - 1) - owner(grp * P.nb) + 1;
    s_slot[0] = owner(grp * P.nb);
  }
  __syncthreads();
  const int nc = s_n, ca = s_slot[0];
  __syncthreads();
  for (int c = ca + r; c < ca + nc; c += blockDim.x)            // slot of the group in CTA c
    s_slot[c - ca] = c * P.maxseg + (int)(grp - (P.units * c / P.ctas) / P.nb);
  __syncthreads();
  const int64_t n = grp * kRowsCta + r;
  const float sw = __ldg(P.w_scales + n);
  asm volatile("griddepcontrol.wait;" ::: "memory");           // the GEMM's partials are complete
  float acc[8] = {};
  constexpr int B = 4;                                          // slots read per batch
  for (int c0 = 0; c0 < nc; c0 += B) {
    float4 v[B][2];
#pragma unroll
    for (int b = 0; b < B; ++b)
      if (c0 + b < nc) {
        const float4* src = reinterpret_cast<const float4*>(P.part + ((int64_t)s_slot[c0 + b] * kRowsCta + r) * 8);
        v[b][0] = __ldcg(src);
        v[b][1] = __ldcg(src + 1);
      }
#pragma unroll
    for (int b = 0; b < B; ++b)
      if (c0 + b < nc) {
        acc[0] += v[b][0].x; acc[1] += v[b][0].y; acc[2] += v[b][0].z; acc[3] += v[b][0].w;
        acc[4] += v[b][1].x; acc[5] += v[b][1].y; acc[6] += v[b][1].z; acc[7] += v[b][1].w;
      }
  }
#pragma unroll
  for (int m = 0; m < 8; ++m) {
    if (m >= P.M) break;
    const float f = acc[m] * sw;
    if (P.ydt == COMET_F32) reinterpret_cast<float*>(P.y)[m * P.ldy + n] = f;
    else if (P.ydt == COMET_BF16) reinterpret_cast<__nv_bfloat16*>(P.y)[m * P.ldy + n] = __float2bfloat16_rn(f);
    else reinterpret_cast<__half*>(P.y)[m * P.ldy + n] = __float2half_rn(f);
  }
}

}  // namespace

int gemv_ctas_per_sm() { return COMET_GEMV_CPS; }
int gemv_stages() { return COMET_GEMV_S; }
constexpr int kStageChoices[3] = {8, 6, 4};   // ring depths instantiated (gemv_pick chooses)

// Plan-time quantities of a grid of `ctas` CTAs: the most groups one CTA touches (workspace
// slots) and the most K-blocks one CTA stages (its shared memory); -1 when that exceeds the
// staging capacity.
int gemv_max_segments(int64_t units, int nb, int ctas) {
  int mx = 1;
  for (int c = 0; c < ctas; ++c) {
    const int64_t u0 = units * c / ctas, u1 = units * (c + 1) / ctas;
    if (u1 > u0) mx = std::max(mx, (int)((u1 - 1) / nb - u0 / nb + 1));
  }
  return mx;
}
size_t gemv_smem_bytes(int64_t M, int nbr, int S) {
  return (size_t)8 * S * 1024 + (size_t)nbr * (M * 128 + 8 * 4 + 4 * 4);
}
// CTAs sharing one row group (the reduction reads at most kMaxRed)
static int gemv_max_group_ctas(int64_t units, int nb, int ctas) {
  const int64_t per = units / ctas;                             // units per CTA, rounded down
  return per <= 0 ? nb : (int)std::min<int64_t>(nb, (nb + per - 1) / per + 1);
}
int gemv_stage_blocks(int64_t units, int nb, int ctas) {
  const int64_t len = (units + ctas - 1) / ctas;
  const int nbr = (int)std::min<int64_t>(nb, len);
  return nbr > kMaxStageBlocks ? -1 : nbr;
}

// Ring depth S and CTAs per SM for this shape: of the (S, CTAs per SM <= COMET_GEMV_CPS) whose
// shared memory fits an SM, the one with the most weight bytes in flight per SM (S x CTAs; ties
// to the deeper ring).  Returns the grid (CTAs), the K-blocks each stages and S; -1 when nothing
// fits.  (The activation staging grows with M: at M = 4 a 6-deep ring at 3 CTAs per SM keeps
// more bytes in flight than an 8-deep one at 2.)
int gemv_pick(int64_t M, int64_t units, int nb, int num_sms, int* nbr_out, int* s_out) {
  int best = -1, best_ctas = -1;
  for (int S : kStageChoices)
    for (int cps = COMET_GEMV_CPS; cps >= 1; --cps) {
      const int ctas = (int)std::min<int64_t>((int64_t)num_sms * cps, units);   // no empty ranges
      const int nbr = gemv_stage_blocks(units, nb, ctas);
      if (nbr < 0 || gemv_max_group_ctas(units, nb, ctas) > kMaxRed) continue;
      if ((size_t)cps * (gemv_smem_bytes(M, nbr, S) + 1024) > (size_t)228 * 1024) continue;
      if (S * cps > best) { best = S * cps; best_ctas = ctas; *nbr_out = nbr; *s_out = S; }
      break;                                                 // fewer CTAs at this S: never better
    }
  return best_ctas;
}

cudaError_t launch_gemv(const uint8_t* w, const uint8_t* codes, const float* scales, const int16_t* qsum,
                        const float* w_scales, void* y, int ydt, int64_t ldy, int64_t M, int64_t N,
                        int64_t K, int64_t Mp, const TagMask& tags, int ctas, int maxseg, int nbr,
                        int S, float* part, cudaStream_t stream, const void* x, int64_t ldx, bool xbf16) {
  VParams P;
  P.w = w; P.codes = codes; P.scales = scales; P.qsum = qsum; P.part = part; P.w_scales = w_scales;
  P.y = y; P.M = M; P.N = N; P.K = K; P.Mp = Mp; P.ldy = ldy;
  P.nb = (int)(K / kBlockK);
  P.units = (N / kRowsCta) * P.nb;
  P.early = N * K / 2 < (64ll << 20) ? 1 : 0;
  P.maxseg = maxseg;
  P.ctas = ctas;
  P.nbr = nbr;
  P.ydt = ydt;
  P.tags = tags;
  P.x = static_cast<const uint16_t*>(x);
  P.ldx = ldx;
  P.xbf16 = xbf16 ? 1 : 0;
  const size_t smem = gemv_smem_bytes(M, nbr, S);
  const bool fq = x != nullptr;
  auto kern = S == 8 ? (fq ? k_gemv<8, true> : k_gemv<8, false>)
            : S == 6 ? (fq ? k_gemv<6, true> : k_gemv<6, false>) : (fq ? k_gemv<4, true> : k_gemv<4, false>);
  // the dynamic shared memory this launch needs (set per device and ring depth when it grows)
  static std::atomic<int> attr_bytes[6][64];
  const int si = (S == 8 ? 0 : S == 6 ? 1 : 2) + (fq ? 3 : 0);
  int dev = 0;
  cudaGetDevice(&dev);
  if ((int)smem > attr_bytes[si][dev & 63].load()) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e == cudaSuccess) e = cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    if (e != cudaSuccess) return e;
    attr_bytes[si][dev & 63].store((int)smem);
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)ctas);
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, kern, P);
  if (e != cudaSuccess) return e;
  cfg.gridDim = dim3((unsigned)(N / kRowsCta));
  cfg.blockDim = dim3(kRowsCta);
  cfg.dynamicSmemBytes = 0;
  return cudaLaunchKernelEx(&cfg, k_gemv_reduce, P);
}

}  // namespace gemv
}  // namespace comet
