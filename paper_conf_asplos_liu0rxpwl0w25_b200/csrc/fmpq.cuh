// fmpq.cuh -- the FMPQ per-(token, block) quantisation arithmetic of kernel 1 (
// readings R1-R5 in DESIGN.md), shared by kernel 1 (quantize.cu) and the decode GEMM's fused
// quantiser (gemm.cu, comet_w4ax_linear): one definition, so both produce the same codes,
// scales and code sums bit for bit.
#pragma once
#include <cstdint>
#include <cuda_fp16.h>
#include <cuda_bf16.h>

namespace comet {
namespace fmpq {

__device__ __forceinline__ uint4 ldg_stream(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p));
  return r;
}

template <bool BF16>
__device__ __forceinline__ void unpack8(const uint4& raw, float (&v)[8]) {
  const uint32_t w[4] = {raw.x, raw.y, raw.z, raw.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    if (BF16) {
      v[2 * i] = __uint_as_float(w[i] << 16);
      v[2 * i + 1] = __uint_as_float(w[i] & 0xFFFF0000u);
    } else {
      __half2 h = *reinterpret_cast<const __half2*>(&w[i]);
      float2 f = __half22float2(h);
      v[2 * i] = f.x;
      v[2 * i + 1] = f.y;
    }
  }
}

// E4M3 byte of an integer q in [-7, 7]: |q| -> {00,38,40,44,48,4A,4C,4E}, sign in bit 7.
__device__ __forceinline__ uint32_t e4m3_of_int4(int q) {
  const uint32_t a = (uint32_t)(q < 0 ? -q : q);
  const uint32_t e = __byte_perm(0x44403800u, 0x4E4C4A48u, a) & 0xFFu;
  return e | (q < 0 ? 0x80u : 0u);
}

// Packed binary32 pairs (FMUL2 / FADD2 on sm_100a), round-to-nearest-even, never contracted.
__device__ __forceinline__ float2 fmul2_rn(float2 a, float2 b) {
  float2 d;
  asm("{\n\t.reg .b64 ra, rb, rd;\n\tmov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\t"
      "mul.rn.f32x2 rd, ra, rb;\n\tmov.b64 {%0, %1}, rd;\n\t}\n"
      : "=f"(d.x), "=f"(d.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
  return d;
}
// a + b as fma(a, 1, b): one rounding, so exactly RN(a + b).  (ptxas contracts a preceding
// mul.rn.f32x2 with add.rn.f32x2 into one FFMA2 -- a single rounding of a*r + b, which breaks
// the tie cases of the definition -- but leaves FMUL2 followed by this FFMA2 alone.)
__device__ __forceinline__ float2 fadd2_rn(float2 a, float2 b) {
  float2 d;
  asm("{\n\t.reg .b64 ra, rb, rc, rd;\n\tmov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%6, %6};\n\t"
      "mov.b64 rc, {%4, %5};\n\tfma.rn.f32x2 rd, ra, rb, rc;\n\tmov.b64 {%0, %1}, rd;\n\t}\n"
      : "=f"(d.x), "=f"(d.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y), "f"(1.0f));
  return d;
}
// E4M3 bytes of two floats (exact for the integers |q| <= 7): low byte <- lo, high byte <- hi.
__device__ __forceinline__ uint32_t e4m3x2(float lo, float hi) {
  uint16_t d;
  asm("cvt.rn.satfinite.e4m3x2.f32 %0, %1, %2;" : "=h"(d) : "f"(hi), "f"(lo));
  return d;
}

// Rounding by the magic constant 1.5 * 2^23: for |t| < 2^22, RN(t + 1.5 * 2^23) =
// 1.5 * 2^23 + rint(t) with rint = round half to even (reading R3), so the low bits of its
// binary32 pattern are the two's-complement integer rint(t) and RN(that - 1.5 * 2^23) is
// rint(t) as a float, exactly.
constexpr float kMagic = 12582912.0f;

// One lane's share of one block: 32 channels (four runs of 8 consecutive channels at
// 32 j + 8 sub, j = 0..3) -- four lanes (sub = 0..3) cover the block's 128 channels.
//   Fast path (every finite r = qmax/amax, and amax == 0): t = x * r as one binary32 product,
//   q = rint(t) by the magic constant.  |x| <= amax gives |t| <= qmax (1 + 2^-24)^2, so
//   rint(t) never exceeds qmax and the clamp of the definition is a no-op.
//   Slow path (a binary32-subnormal amax, where qmax/amax overflows to inf, reading R5):
//   the definition written out with a saturating conversion and the clamp.
struct LaneOut {
  uint2 c[4];        // 4 x 8 code bytes
  float s;           // block scale (same in the 4 lanes)
  int q;             // block code sum (same in the 4 lanes, after the reduction)
};

__device__ __forceinline__ LaneOut quantize32(const float (&v)[32], bool is8) {
  float a = 0.f;
#pragma unroll
  for (int j = 0; j < 32; ++j) a = fmaxf(a, fabsf(v[j]));
  a = fmaxf(a, __shfl_xor_sync(0xffffffffu, a, 1));
  a = fmaxf(a, __shfl_xor_sync(0xffffffffu, a, 2));
  const float qmax = is8 ? 127.f : 7.f;
  LaneOut o;
  o.s = (a == 0.f) ? 0.f : __fdiv_rn(a, qmax);
  const float r = __fdiv_rn(qmax, a);          // +inf for an all-zero block
  float qsf = 0.f;
  int qsi = 0;
  if (a == 0.f || r <= 3.0e38f) {
    const float rr = a == 0.f ? 0.f : r;       // zero block: every code 0
    float2 acc = make_float2(0.f, 0.f);
    if (is8) {
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        uint32_t p[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float2 y = fadd2_rn(fmul2_rn(make_float2(v[8 * j + 2 * i], v[8 * j + 2 * i + 1]), make_float2(rr, rr)),
                                    make_float2(kMagic, kMagic));
          acc = fadd2_rn(acc, fadd2_rn(y, make_float2(-kMagic, -kMagic)));
          // two's-complement byte of rint(t) = low byte of the biased pattern
          p[i] = __byte_perm(__float_as_uint(y.x), __float_as_uint(y.y), 0x0040);
        }
        o.c[j] = make_uint2(__byte_perm(p[0], p[1], 0x5410), __byte_perm(p[2], p[3], 0x5410));
      }
    } else {
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        uint32_t e[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float2 y = fadd2_rn(fmul2_rn(make_float2(v[8 * j + 2 * i], v[8 * j + 2 * i + 1]), make_float2(rr, rr)),
                                    make_float2(kMagic, kMagic));
          const float2 f = fadd2_rn(y, make_float2(-kMagic, -kMagic));   // rint(t), +0 for 0
          acc = fadd2_rn(acc, f);
          e[i] = e4m3x2(f.x, f.y);
        }
        o.c[j] = make_uint2(e[0] | (e[1] << 16), e[2] | (e[3] << 16));
      }
    }
    qsf = acc.x + acc.y;                       // integers < 2^13: exact
  } else {
    const int iq = is8 ? 127 : 7;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      uint32_t bytes[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        const float t = __fmul_rn(v[8 * j + i], r);
        int q = __float2int_rn(t);              // cvt.rni.s32.f32: half-even, NaN -> 0, saturating
        q = min(max(q, -iq), iq);
        qsi += q;
        bytes[i] = is8 ? ((uint32_t)q & 0xFFu) : e4m3_of_int4(q);
      }
      o.c[j] = make_uint2(bytes[0] | (bytes[1] << 8) | (bytes[2] << 16) | (bytes[3] << 24),
                          bytes[4] | (bytes[5] << 8) | (bytes[6] << 16) | (bytes[7] << 24));
    }
  }
  int qs = qsi + (int)qsf;
  qs += __shfl_xor_sync(0xffffffffu, qs, 1);
  qs += __shfl_xor_sync(0xffffffffu, qs, 2);
  o.q = qs;
  return o;
}

}  // namespace fmpq
}  // namespace comet
