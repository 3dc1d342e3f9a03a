// gemm_common.cuh -- pieces shared by the two W4Ax GEMM kernels (gemm.cu: weights on the MMA M
// side, for decode-sized token counts; gemm_n.cu: tokens on the MMA M side, for prefill).
#pragma once
#include <cudaTypedefs.h>
#include <cuda_fp16.h>
#include <cuda_bf16.h>
#include "internal.h"
#include "sm100.cuh"

namespace comet {
namespace gemm {

using namespace sm100;

constexpr int kThreads = 512;

struct __align__(64) GemmParams {
  CUtensorMap map_x;
  CUtensorMap map_w;
  CUtensorMap map_y;         // prefill kernel: Y as bytes [M][N*esz], box 64 B x 128 rows (32 rows
                             // with COMET_EPI_WARP), 64B swizzle
  CUtensorMap map_s;         // decode kernel: act_scales [nb][Mp] f32, box NT x KS
  CUtensorMap map_q;         // decode kernel, grouped scales: qsum [nb][Mp] int16, box NT x KS
  CUtensorMap map_g;         // decode kernel, grouped scales: s_w [nb][N] f32, box 128 x KS
  const float* scales;       // [nb][Mp]
  const float* corr;         // [Mp]
  const int16_t* qsum;       // [nb][Mp]
  const float* w_scales;     // [N]
  void* y;
  int64_t ldy;
  int32_t* dbg_acc;          // [M][N] or null
  int32_t* dbg_blocks;       // [nb][M][N] or null
  float* ws_part;
  uint32_t* ws_flags;
  const int32_t* cta_begin;
  const WorkItem* items;
  int64_t M, N, Mp;
  int nb, n_m_tiles, max_seg, ydt;
  uint32_t epoch;
  unsigned long long* trace;  // diagnostic only (comet_debug_set_trace): [cta<2][event<8][kb<1024] clock64
  int ablate;                // diagnostic only (env COMET_ABLATE): 4 skip widening, 8 skip MMAs
                             // (prefill kernel); the output is invalid under it
  // NEXT-2 fused reduce-scatter (prefill pair kernel): when rs_world > 0 the epilogue stores
  // this rank's FP32 partial of output row m straight into the receive buffer of the rank that
  // owns row m (P2P over NVLink; owner = m / rs_ms), slot [rs_rank][m - owner * rs_ms][N]
  int rs_world, rs_rank;
  int64_t rs_ms;
  float* rs_dst[8];
  TagMask tags;
  // FQ (fused quantiser, comet_w4ax_linear): the 16-bit input x [M][ldxq] read by the decode
  // kernel's quantiser warps instead of TMA-loaded codes
  const void* xq;
  int64_t ldxq;
  int xq_bf16;
};

// Widening of packed INT4 weights (the B200 form of the paper's "location switch" + "zero
// extension"; layout R14 in include/comet.h).  One packed 32-bit word holds 8
// consecutive channels; widen_int4 yields their offset-binary bytes u = w + 8 in channel order
// (lo = channels 0..3, hi = 4..7) in 3 instructions -- the byte u read as E4M3 is exactly
// u * 2^-9, the INT4-block MMA operand.  int4_to_int8 turns such a word into the s8 bytes 16 w
// = (u << 4) ^ 0x80 of an INT8 block.  Every GEMM kernel widens through these two functions;
// comet_debug_widen runs them on caller-chosen words (exhaustive pin I9).
__device__ __forceinline__ void widen_int4(uint32_t pv, uint32_t& lo, uint32_t& hi) {
  lo = pv & 0x0F0F0F0Fu;
  hi = (pv >> 4) & 0x0F0F0F0Fu;
}
__device__ __forceinline__ uint32_t int4_to_int8(uint32_t u4) { return (u4 << 4) ^ 0x80808080u; }
// One K-block row of a weight (64 packed bytes = 4 x uint4) -> 128 widened bytes (32 words) in
// channel order.  The block kind is a template parameter: the caller branches once per K-block
// (warp-uniform), so an INT4 block costs exactly the 3 instructions per 8 values of widen_int4
// (a runtime flag inside the loop gets if-converted: both forms computed and selected per word).
template <bool IS8>
__device__ __forceinline__ void widen_kblock_row(const uint4* c, uint32_t (&o)[32]) {
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const uint32_t pw[4] = {c[j].x, c[j].y, c[j].z, c[j].w};
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const int g = 2 * (j * 4 + e);
      widen_int4(pw[e], o[g], o[g + 1]);
      if (IS8) {
        o[g] = int4_to_int8(o[g]);
        o[g + 1] = int4_to_int8(o[g + 1]);
      }
    }
  }
}

// Packed binary32 pairs, round-to-nearest (FMUL2 / FADD2 on sm_100a).
__device__ __forceinline__ float2 fmul2_f(float2 a, float2 b) {
  float2 d;
  asm("{\n\t.reg .b64 ra, rb, rd;\n\tmov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\t"
      "mul.rn.f32x2 rd, ra, rb;\n\tmov.b64 {%0, %1}, rd;\n\t}\n"
      : "=f"(d.x), "=f"(d.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
  return d;
}
__device__ __forceinline__ float2 fadd2_f(float2 a, float2 b) {
  float2 d;
  asm("{\n\t.reg .b64 ra, rb, rd;\n\tmov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\t"
      "add.rn.f32x2 rd, ra, rb;\n\tmov.b64 {%0, %1}, rd;\n\t}\n"
      : "=f"(d.x), "=f"(d.y) : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
  return d;
}

// Exact int32 -> binary32 of two INT8-block accumulators (|v| <= 16 * 128 * 127 * 8 =
// 2,080,768 < 2^22).  Default: two I2F.  COMET_I2F_MAGIC=1 instead adds 0x4B400000 (the bit
// pattern of 1.5 * 2^23 + v) and subtracts 1.5 * 2^23 with one exact packed FMA -- no I2F, but
// measured slower in the prefill promotion (tools/fsweep.py, all-INT8 blocks: 1556 against
// 1805 TOPS on the same box), so it is off.
#ifndef COMET_I2F_MAGIC
#define COMET_I2F_MAGIC 0
#endif
__device__ __forceinline__ float2 i2f2_exact(uint32_t a, uint32_t b) {
  if (!COMET_I2F_MAGIC) return make_float2(__int2float_rn((int)a), __int2float_rn((int)b));
  const float2 x = make_float2(__uint_as_float(a + 0x4B400000u), __uint_as_float(b + 0x4B400000u));
  return ffma2(x, make_float2(1.f, 1.f), make_float2(-12582912.f, -12582912.f));
}

// A global load the compiler keeps where it is written (volatile) and whose result is consumed
// only where the caller first uses it: for operands prefetched a work item ahead.
__device__ __forceinline__ float ldg_nc_f32(const float* p) {
  float v;
  asm volatile("ld.global.nc.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}

__device__ __forceinline__ void named_bar_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ void st_release_gpu(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void fence_acq_rel_gpu() {
  asm volatile("fence.acq_rel.gpu;" ::: "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
template <uint32_t N>
__device__ __forceinline__ void setmaxnreg_dec() {
  asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(N));
}
template <uint32_t N>
__device__ __forceinline__ void setmaxnreg_inc() {
  asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(N));
}

__device__ __forceinline__ WorkItem load_item(const GemmParams& P, int idx, bool debug) {
  if (debug) {
    WorkItem w{};
    w.tile = idx; w.kb_begin = 0; w.kb_end = P.nb; w.flags = 2; w.fix = -1;
    return w;
  }
  const int4* src = reinterpret_cast<const int4*>(P.items + idx);
  int4 a = __ldg(src);
  int4 b = __ldg(src + 1);
  WorkItem w;
  w.tile = a.x; w.kb_begin = a.y; w.kb_end = a.z; w.flags = a.w;
  w.fix = b.x; w.pad0 = b.y; w.pad1 = b.z; w.pad2 = b.w;
  return w;
}

// Diagnostic hooks (timeline trace, stage ablation) exist only in a COMET_DIAG=1 build.
#ifndef COMET_DIAG
#define COMET_DIAG 0
#endif
#ifndef COMET_TRACE
#define COMET_TRACE 0       // 1: timeline trace only (tools/trace_gemm.py), no ablation hooks
#endif
#ifndef COMET_EPI_WARP
#define COMET_EPI_WARP 1   // prefill epilogue: every warp stores its own 32 rows (no warpgroup barriers)
#endif
#ifndef COMET_ABLATE_CT
#define COMET_ABLATE_CT 0   // compile-time ablation bits (timing experiments only; wrong results)
#endif
__device__ __forceinline__ int diag_ablate(const GemmParams& P) {
  return (COMET_DIAG ? P.ablate : 0) | COMET_ABLATE_CT;
}

// Diagnostic timeline: CTA c < 2, event e < 8, K-block index i < 1024 (per-CTA running count).
#ifndef COMET_TRACE_MASK
#define COMET_TRACE_MASK 0xFFFF   // events recorded by a trace build (bit e = event e)
#endif
__device__ __forceinline__ void trace_ev(const GemmParams& P, int e, int i) {
  if ((COMET_DIAG || COMET_TRACE) && ((COMET_TRACE_MASK >> e) & 1) && P.trace != nullptr && blockIdx.x < 2 && i < 1024) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%clock64;" : "=l"(t));
    P.trace[((int)blockIdx.x * 16 + e) * 1024 + i] = t;
  }
}

// Host: TMA descriptor helpers (gemm.cu).
bool make_map_2d(CUtensorMap* map, const void* base, uint64_t inner, uint64_t outer,
                 uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer, CUtensorMapSwizzle swz);
// General tiled map: `rank` dims (innermost first), byte strides of dims 1.. , box sizes.
bool make_map(CUtensorMap* map, CUtensorMapDataType dt, int rank, const void* base,
              const uint64_t* dims, const uint64_t* stride_bytes, const uint32_t* box,
              CUtensorMapSwizzle swz);

extern unsigned long long* g_trace;   // diagnostic timeline buffer (comet_debug_set_trace)

// Stream-K fix-up epoch: one process-wide monotonic counter, so no two launches (of any plan,
// on any workspace) publish or wait for the same flag value; a zeroed workspace never matches.
uint32_t next_epoch();

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once per (kernel, device): function
// attributes are per device context, so the flag is a per-device bit (devices 0..63).
template <typename Kern>
inline cudaError_t set_smem_attr(Kern kernel, int bytes, std::atomic<uint64_t>& done) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  const uint64_t bit = 1ull << (dev & 63);
  if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
  if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_acq_rel);
  return e;
}

// Normal-orientation launcher (gemm_n.cu).  BN = weights per tile (256, or 128 for debug);
// cg = CTAs per tile (1, or 2 for the tcgen05 CTA pair; grid must then be even).
cudaError_t launch_gemm_n(const GemmParams& prm, int grid, int bn, int cg, int debug, cudaStream_t stream,
                          bool grouped = false);
// Persistent units (CTAs, or pairs for cg = 2) of the production kernel that fit on the device
// at once (occupancy query; -1 on error).
int max_units_gemm_n(int bn, int cg, int sms);
int stages_gemm_n(int bn, int cg);   // pipeline slots S of the production kernel

}  // namespace gemm
}  // namespace comet
