// kv4.cu -- NEXT-4: INT4 KV-cache quantisation, the "KV4" of W4A4KV4.
//
// P:L146 "a channel-wise 4-bit quantization strategy for the KV cache"; "channel-wise
// asymmetric INT4 group quantization for the KV cache"; reading R17: a K or V
// cache tensor X[T][C] (C = KV heads x head_dim) is quantised per (group of G consecutive
// tokens, channel) with an asymmetric min-max quantiser, in binary32, never contracted:
//   mn = min x, mx = max x, d = mx - mn, s = d/15, r = 15/d (d == 0: s = r = 0),
//   q = clamp(rint((x - mn) * r), 0, 15);   x_hat = mn + q * s (two roundings) -> f16/bf16.
// Both kernels are HBM-bound (2 B in + 0.5 B out per element, and the reverse).
//
// Quantise: a CTA owns G tokens x 64 channels.  Thread (row slot j = tid/8, chunk c = tid%8)
// loads rows j, j+32, ... (16 B = 8 channels each, all loads in flight at once, kept in
// registers), reduces min/max over its rows, then over the 4 lanes of its warp that share the
// chunk (xor 8, 16) and over the 8 warps through shared memory; then quantises its registers
// and writes 4 code bytes per row (8 threads = 32 contiguous bytes per row).
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include <cfloat>
#include "internal.h"

namespace comet {
namespace {

template <bool BF16>
__device__ __forceinline__ void unpack8f(const uint4& raw, float (&v)[8]) {
  const uint32_t w[4] = {raw.x, raw.y, raw.z, raw.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    if (BF16) {
      v[2 * i] = __uint_as_float(w[i] << 16);
      v[2 * i + 1] = __uint_as_float(w[i] & 0xFFFF0000u);
    } else {
      const float2 f = __half22float2(*reinterpret_cast<const __half2*>(&w[i]));
      v[2 * i] = f.x;
      v[2 * i + 1] = f.y;
    }
  }
}

// Packed binary32 pairs, each one correctly rounded operation (never contracted: an FFMA2 by
// +-1 is a single rounding of the sum, and ptxas leaves FMUL2 -> FFMA2 chains alone).
__device__ __forceinline__ float2 ffma2_rn(float2 a, float2 b, float2 c) {
  float2 d;
  asm("{\n\t.reg .b64 ra, rb, rc, rd;\n\tmov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\t"
      "mov.b64 rc, {%6, %7};\n\tfma.rn.f32x2 rd, ra, rb, rc;\n\tmov.b64 {%0, %1}, rd;\n\t}\n"
      : "=f"(d.x), "=f"(d.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y), "f"(c.x), "f"(c.y));
  return d;
}
__device__ __forceinline__ float2 fmul2_rn(float2 a, float2 b) {
  float2 d;
  asm("{\n\t.reg .b64 ra, rb, rd;\n\tmov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\t"
      "mul.rn.f32x2 rd, ra, rb;\n\tmov.b64 {%0, %1}, rd;\n\t}\n"
      : "=f"(d.x), "=f"(d.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
  return d;
}
// min / max of two packed 16-bit pairs (exact in the input format: no conversion needed)
template <bool BF16>
__device__ __forceinline__ uint32_t min2(uint32_t a, uint32_t b) {
  uint32_t d;
  if (BF16) asm("min.bf16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  else asm("min.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
template <bool BF16>
__device__ __forceinline__ uint32_t max2(uint32_t a, uint32_t b) {
  uint32_t d;
  if (BF16) asm("max.bf16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  else asm("max.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
template <bool BF16>
__device__ __forceinline__ float2 to_f2(uint32_t w) {
  if (BF16) return make_float2(__uint_as_float(w << 16), __uint_as_float(w & 0xFFFF0000u));
  return __half22float2(*reinterpret_cast<const __half2*>(&w));
}

template <bool BF16, int RPT>   // RPT = rows per thread = G / 32
__global__ void __launch_bounds__(256, 4) k_kv4_quantize(const uint16_t* __restrict__ x, int64_t T,
                                                      int64_t C, int64_t ldx, int G,
                                                      uint8_t* __restrict__ codes,
                                                      float* __restrict__ scales,
                                                      float* __restrict__ mins) {
  __shared__ float s_lo[8][64], s_hi[8][64];
  __shared__ __align__(16) float s_mn[64], s_r[64];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int j = tid >> 3, ch = tid & 7;
  const int64_t g = blockIdx.y;
  const int64_t c0 = (int64_t)blockIdx.x * 64 + ch * 8;
  const int64_t t0 = g * G;
  uint4 raw[RPT];
#pragma unroll
  for (int i = 0; i < RPT; ++i) {
    const int64_t t = t0 + j + 32 * i;
    raw[i] = (t < T && 32 * i + j < G) ? __ldg(reinterpret_cast<const uint4*>(x + t * ldx + c0))
                                       : make_uint4(0, 0, 0, 0);
  }
  // pass 1: min / max on the packed 16-bit pairs (row slot 0 always holds a valid row)
  uint32_t lo2[4] = {raw[0].x, raw[0].y, raw[0].z, raw[0].w};
  uint32_t hi2[4] = {raw[0].x, raw[0].y, raw[0].z, raw[0].w};
#pragma unroll
  for (int i = 1; i < RPT; ++i) {
    const int64_t t = t0 + j + 32 * i;
    if (t < T && 32 * i + j < G) {
      const uint32_t w[4] = {raw[i].x, raw[i].y, raw[i].z, raw[i].w};
#pragma unroll
      for (int e = 0; e < 4; ++e) { lo2[e] = min2<BF16>(lo2[e], w[e]); hi2[e] = max2<BF16>(hi2[e], w[e]); }
    }
  }
  if (t0 + j >= T) {                                   // this slot has no row: neutral values
#pragma unroll
    for (int e = 0; e < 4; ++e) { lo2[e] = BF16 ? 0x7F7F7F7Fu : 0x7BFF7BFFu; hi2[e] = BF16 ? 0xFF7FFF7Fu : 0xFBFFFBFFu; }
  }
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    lo2[e] = min2<BF16>(lo2[e], __shfl_xor_sync(0xffffffffu, lo2[e], 8));
    lo2[e] = min2<BF16>(lo2[e], __shfl_xor_sync(0xffffffffu, lo2[e], 16));
    hi2[e] = max2<BF16>(hi2[e], __shfl_xor_sync(0xffffffffu, hi2[e], 8));
    hi2[e] = max2<BF16>(hi2[e], __shfl_xor_sync(0xffffffffu, hi2[e], 16));
  }
  float lo[8], hi[8];
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    const float2 l = to_f2<BF16>(lo2[e]), h = to_f2<BF16>(hi2[e]);
    lo[2 * e] = l.x; lo[2 * e + 1] = l.y; hi[2 * e] = h.x; hi[2 * e + 1] = h.y;
  }
  if (lane < 8) {
#pragma unroll
    for (int e = 0; e < 8; ++e) { s_lo[warp][ch * 8 + e] = lo[e]; s_hi[warp][ch * 8 + e] = hi[e]; }
  }
  __syncthreads();
  // one thread per channel finishes the reduction and the two divisions
  if (tid < 64) {
    float a = s_lo[0][tid], b = s_hi[0][tid];
#pragma unroll
    for (int w = 1; w < 8; ++w) { a = fminf(a, s_lo[w][tid]); b = fmaxf(b, s_hi[w][tid]); }
    const float d = __fsub_rn(b, a);
    s_mn[tid] = a;
    s_r[tid] = d == 0.f ? 0.f : __fdiv_rn(15.f, d);
    const int64_t c = (int64_t)blockIdx.x * 64 + tid;
    scales[g * C + c] = d == 0.f ? 0.f : __fdiv_rn(d, 15.f);
    mins[g * C + c] = a;
  }
  __syncthreads();
  float mn[8], r[8];
  {
    const float4 a0 = *reinterpret_cast<const float4*>(&s_mn[ch * 8]);
    const float4 a1 = *reinterpret_cast<const float4*>(&s_mn[ch * 8 + 4]);
    const float4 b0 = *reinterpret_cast<const float4*>(&s_r[ch * 8]);
    const float4 b1 = *reinterpret_cast<const float4*>(&s_r[ch * 8 + 4]);
    mn[0] = a0.x; mn[1] = a0.y; mn[2] = a0.z; mn[3] = a0.w; mn[4] = a1.x; mn[5] = a1.y; mn[6] = a1.z; mn[7] = a1.w;
    r[0] = b0.x; r[1] = b0.y; r[2] = b0.z; r[3] = b0.w; r[4] = b1.x; r[5] = b1.y; r[6] = b1.z; r[7] = b1.w;
  }
#pragma unroll
  for (int i = 0; i < RPT; ++i) {
    const int64_t t = t0 + j + 32 * i;
    if (t < T && 32 * i + j < G) {
      const uint32_t w[4] = {raw[i].x, raw[i].y, raw[i].z, raw[i].w};
      uint32_t word = 0;
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        // 0 <= (x - mn) * r <= 15 (1 + 2^-23)^2, so rint lands in [0, 15] and the clamp of the
        // definition never acts; rint (half-even) by the magic constant 1.5 * 2^23.  Pairs:
        // RN(x - mn) = fma(mn, -1, x), RN(. * r), RN(. + magic) = fma(., 1, magic).
        const float2 v = to_f2<BF16>(w[e]);
        const float2 d = ffma2_rn(make_float2(mn[2 * e], mn[2 * e + 1]), make_float2(-1.f, -1.f), v);
        const float2 tq = fmul2_rn(d, make_float2(r[2 * e], r[2 * e + 1]));
        const float2 y = ffma2_rn(tq, make_float2(1.f, 1.f), make_float2(12582912.0f, 12582912.0f));
        word |= ((__float_as_uint(y.x) & 0xFu) | ((__float_as_uint(y.y) & 0xFu) << 4)) << (8 * e);
      }
      *reinterpret_cast<uint32_t*>(codes + t * (C / 2) + c0 / 2) = word;
    }
  }
}

// Dequantise: thread = (4 consecutive tokens of one group, 8 channels): four 32-bit code loads
// issued together, the group's 8 scales and mins once (L1/L2-resident across the group's
// tokens), four 16-byte stores.  Groups are multiples of 4 tokens, so the 4 rows share them.
template <bool BF16>
__global__ void __launch_bounds__(256) k_kv4_dequantize(const uint8_t* __restrict__ codes,
                                                        const float* __restrict__ scales,
                                                        const float* __restrict__ mins, int64_t T,
                                                        int64_t C, int G, uint16_t* __restrict__ y,
                                                        int64_t ldy) {
  const int64_t chunks = C / 8;
  const int64_t n = ((T + 3) / 4) * chunks;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t t0 = (i / chunks) * 4, c0 = (i % chunks) * 8, g = t0 / G;
    uint32_t word[4];
#pragma unroll
    for (int r = 0; r < 4; ++r)
      word[r] = t0 + r < T ? __ldg(reinterpret_cast<const uint32_t*>(codes + (t0 + r) * (C / 2) + c0 / 2)) : 0u;
    const float4 s0 = __ldg(reinterpret_cast<const float4*>(scales + g * C + c0));
    const float4 s1 = __ldg(reinterpret_cast<const float4*>(scales + g * C + c0 + 4));
    const float4 m0 = __ldg(reinterpret_cast<const float4*>(mins + g * C + c0));
    const float4 m1 = __ldg(reinterpret_cast<const float4*>(mins + g * C + c0 + 4));
    const float sv[8] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
    const float mv[8] = {m0.x, m0.y, m0.z, m0.w, m1.x, m1.y, m1.z, m1.w};
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      if (t0 + r >= T) break;
      uint32_t out[4];
#pragma unroll
      for (int e = 0; e < 8; e += 2) {
        const float a = __fadd_rn(mv[e], __fmul_rn((float)((word[r] >> (4 * e)) & 0xFu), sv[e]));
        const float b = __fadd_rn(mv[e + 1], __fmul_rn((float)((word[r] >> (4 * e + 4)) & 0xFu), sv[e + 1]));
        if (BF16) {
          const __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
          out[e / 2] = *reinterpret_cast<const uint32_t*>(&h);
        } else {
          const __half2 h = __floats2half2_rn(a, b);
          out[e / 2] = *reinterpret_cast<const uint32_t*>(&h);
        }
      }
      *reinterpret_cast<uint4*>(y + (t0 + r) * ldy + c0) = make_uint4(out[0], out[1], out[2], out[3]);
    }
  }
}

}  // namespace

cudaError_t launch_kv4_quantize(const void* x, bool bf16, int64_t T, int64_t C, int64_t ldx, int G,
                                uint8_t* codes, float* scales, float* mins, cudaStream_t stream) {
  const dim3 grid((unsigned)(C / 64), (unsigned)ceil_div(T, G));
  const uint16_t* xp = static_cast<const uint16_t*>(x);
#define COMET_KV4_Q(RPT)                                                                              \
  (bf16 ? (k_kv4_quantize<true, RPT><<<grid, 256, 0, stream>>>(xp, T, C, ldx, G, codes, scales, mins), 0) \
        : (k_kv4_quantize<false, RPT><<<grid, 256, 0, stream>>>(xp, T, C, ldx, G, codes, scales, mins), 0))
  switch (G) {
    case 32: COMET_KV4_Q(1); break;
    case 64: COMET_KV4_Q(2); break;
    case 128: COMET_KV4_Q(4); break;
    default: COMET_KV4_Q(8); break;    // 256
  }
#undef COMET_KV4_Q
  return cudaGetLastError();
}

cudaError_t launch_kv4_dequantize(const uint8_t* codes, const float* scales, const float* mins,
                                  int64_t T, int64_t C, int G, void* y, bool bf16, int64_t ldy,
                                  cudaStream_t stream) {
  const int64_t n = ceil_div(T, 4) * (C / 8);
  const int64_t blocks = std::min<int64_t>(ceil_div(n, 256), 148 * 16);
  uint16_t* yp = static_cast<uint16_t*>(y);
  if (bf16) k_kv4_dequantize<true><<<(unsigned)blocks, 256, 0, stream>>>(codes, scales, mins, T, C, G, yp, ldy);
  else k_kv4_dequantize<false><<<(unsigned)blocks, 256, 0, stream>>>(codes, scales, mins, T, C, G, yp, ldy);
  return cudaGetLastError();
}

}  // namespace comet
