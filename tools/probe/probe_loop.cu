// probe_loop.cu -- the prefill pair kernel's MMA <-> promotion loop in isolation.
//
// Static operands in shared memory (no TMA, no widening): one issuing thread runs K-blocks of
// four K=32 MMAs into NACC TMEM accumulators of N columns, commits each K-block to acc_full[a];
// NPW promotion warpgroups per CTA wait acc_full[a], optionally read the accumulator (WORK = 1:
// 64-column rounds of two 32x32b.x32 loads + FFMA2 into register sums, as the production
// promotion), and arrive on ready[a] (in the even CTA), which the issuer waits before reusing
// accumulator a.  Prints clk per K-block for each configuration, so the handshake latency
// (commit -> wake -> arrive -> issue) and the TMEM read cost can be separated.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 probe_loop.cu -o probe_loop
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"
using namespace comet::sm100;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

// wait flavours: 0 production mbar_wait (test_wait, then try_wait with a suspend hint),
// 1 test_wait spin, 2 plain try_wait loop (no hint)
// 3 try_wait with a 1 ms suspend hint, no test_wait first; 4 the same with a 20 us hint;
// 5 test_wait first, then plain try_wait (the production wait at COMET_WAIT_MODE=1, no timer)
__device__ __forceinline__ bool try_wait_hint(uint32_t bar, uint32_t parity, uint32_t ns) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2, %3;\n\tselp.b32 %0, 1, 0, P;\n\t}\n"
               : "=r"(ok) : "r"(bar), "r"(parity), "r"(ns) : "memory");
  return ok != 0;
}
__device__ __forceinline__ bool test_wait1(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred P;\n\tmbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n\tselp.b32 %0, 1, 0, P;\n\t}\n"
               : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
  return ok != 0;
}
template <int W>
__device__ __forceinline__ void wait_k(uint64_t* bar, uint32_t ph) {
  if (W == 0) mbar_wait(bar, ph);
  else if (W == 1) mbar_wait_spin(bar, ph);
  else if (W == 2) { while (!mbar_try_wait(smem_u32(bar), ph)) {} }
  else if (W == 3) { while (!try_wait_hint(smem_u32(bar), ph, 1000000u)) {} }
  else if (W == 4) { while (!try_wait_hint(smem_u32(bar), ph, 20000u)) {} }
  else { if (!test_wait1(smem_u32(bar), ph)) while (!mbar_try_wait(smem_u32(bar), ph)) {} }
}
__device__ __forceinline__ void named_sync(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

// ARR 0: every promotion warp arrives (lane 0); 1: one arrive per CTA after a named barrier.
// NOWAIT: the issuer never waits (pure MMA throughput into one accumulator).
// LOAD 1: warp 0 streams 8 KB bulk copies from an L2-resident buffer (3 per K-block, the
// production kernel's 24 KB of TMA per CTA per K-block) into four smem buffers, concurrently;
// LOAD 2: the same without MMAs (the copy stream alone).
template <int CG, int N, int NACC, int WORK, int SPIN, int ARR, int NPW, int NOWAIT, int LOAD = 0>
__global__ void __launch_bounds__(128 * (1 + NPW), 1) k_loop(int iters, float* out, unsigned long long* cyc,
                                                           const uint8_t* gsrc, unsigned long long* cyc2) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  constexpr int WROWS = N / CG;
  uint8_t* sA = smem;                       // 128 x 128 B
  uint8_t* sB = smem + 16384;               // WROWS x 128 B
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + 16384 + WROWS * 128);
  uint64_t* acc_full = bars;                // [NACC]
  uint64_t* ready = bars + NACC;            // [NACC] (even CTA)
  uint64_t* lbar = bars + 2 * NACC;        // [4] loader
  uint32_t* holder = reinterpret_cast<uint32_t*>(bars + 2 * NACC + 4);
  uint8_t* sL = smem + 16384 + WROWS * 128 + 1024;   // [4][8 KB] loader buffers
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = CG == 2 ? cluster_ctarank() : 0;
  constexpr uint32_t kArrivals = (ARR == 0 ? 4 * NPW : 1) * CG;
  for (int i = threadIdx.x; i < 16384 + WROWS * 128; i += blockDim.x) smem[i] = (uint8_t)((i * 37 + 11) & 0x77);
  if (threadIdx.x == 0) {
    for (int i = 0; i < 4; ++i) mbar_init(&lbar[i], 1);
    for (int i = 0; i < NACC; ++i) { mbar_init(&acc_full[i], 1); mbar_init(&ready[i], kArrivals); mbar_arrive_count(&ready[i], kArrivals); }
    fence_mbar_init();
  }
  if (warp == 2) {
    if (CG == 2) { tmem_alloc_cg2<512>(holder); tmem_relinquish_cg2(); }
    else { tmem_alloc<512>(holder); tmem_relinquish(); }
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  if (CG == 2) cluster_sync();
  tc_fence_after();
  const uint32_t tb = *holder;
  const uint32_t ready_lead = CG == 2 ? mapa_shared(smem_u32(ready), 0) : smem_u32(ready);
  float keep = 0.f;
  if (LOAD && warp == 0) {
    if (lane == 0) {
      const int nl = 3 * iters;
      constexpr int kChunks = (64 << 20) / 8192;
      unsigned long long c0 = clock64();
      for (int i = 0; i < nl; ++i) {
        const int b = i & 3;
        if (i >= 4) mbar_wait(&lbar[b], (uint32_t)((i / 4) - 1) & 1u);
        mbar_arrive_expect_tx(&lbar[b], 8192);
        bulk_load(sL + b * 8192, gsrc + (size_t)(((unsigned)blockIdx.x * 977u + (unsigned)i * 13u) % kChunks) * 8192, 8192, &lbar[b]);
      }
      for (int i = nl; i < nl + 4; ++i) if (i >= 4) mbar_wait(&lbar[i & 3], (uint32_t)((i / 4) - 1) & 1u);
      cyc2[blockIdx.x] = clock64() - c0;
    }
  } else if (warp == 1 && rank == 0 && LOAD == 2) {
    cyc[blockIdx.x] = 1;
  } else if (warp == 1 && rank == 0) {
    const uint32_t id = idesc_i8(128 * CG, N);
    const uint32_t sa = smem_u32(sA), sb = smem_u32(sB);
    unsigned long long c0 = clock64();
    for (int j = 0; j < iters; ++j) {
      const int a = j % NACC;
      const uint32_t ph = (uint32_t)(j / NACC) & 1u;
      if (!NOWAIT) wait_k<SPIN % 8>(&ready[a], ph);
      tc_fence_after();
      if (elect_one()) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const uint64_t ad = sdesc_kmajor_sw128(sa + 32 * k), bd = sdesc_kmajor_sw128(sb + 32 * k);
          if (CG == 2) mma_i8_ss_cg2(tb + (NOWAIT ? 0 : a * N), ad, bd, id, k);
          else mma_i8_ss(tb + (NOWAIT ? 0 : a * N), ad, bd, id, k);
        }
        if (CG == 2) tc_commit_mc(&acc_full[a], 3); else tc_commit(&acc_full[a]);
      }
      __syncwarp();
    }
    if (NOWAIT) {   // drain
      const int a = (iters - 1) % NACC;
      mbar_wait(&acc_full[a], (uint32_t)((iters - 1) / NACC) & 1u);
    }
    unsigned long long c1 = clock64();
    if (lane == 0) cyc[blockIdx.x] = c1 - c0;
  } else if (warp >= 4 && !NOWAIT && LOAD != 2) {
    const int wg = (warp - 4) >> 2, q = warp & 3;
    constexpr int COLS = N / NPW;
    float acc[WORK ? COLS : 1];
#pragma unroll
    for (int c = 0; c < (WORK ? COLS : 1); ++c) acc[c] = 0.f;
    const uint32_t taddr0 = tb + ((uint32_t)(q * 32) << 16) + wg * COLS;
    for (int j = 0; j < iters; ++j) {
      const int a = j % NACC;
      const uint32_t ph = (uint32_t)(j / NACC) & 1u;
      wait_k<SPIN / 8>(&acc_full[a], ph);
      tc_fence_after();
      const float s = 1.0f + 1e-7f * j;
      const float2 s2 = make_float2(s, s);
      if (WORK) {
        constexpr int R = (COLS >= 64 && NPW < 4) ? 64 : 16;
#pragma unroll
        for (int b = 0; b < COLS / R; ++b) {
          uint32_t v[R];
          tmem_ld_32x32b<R>(taddr0 + a * N + b * R, v);
          tmem_wait_ld();
          if (b + 1 == COLS / R) {
            tc_fence_before();
            if (ARR == 0) { __syncwarp(); if (lane == 0) mbar_arrive_cluster(ready_lead + a * 8); }
            else { named_sync(1, 128 * NPW); if (threadIdx.x == 128) mbar_arrive_cluster(ready_lead + a * 8); }
          }
#pragma unroll
          for (int c = 0; c < R; c += 2) {
            const float2 y = ffma2(make_float2(__uint_as_float(v[c]), __uint_as_float(v[c + 1])), s2,
                                   make_float2(acc[b * R + c], acc[b * R + c + 1]));
            acc[b * R + c] = y.x; acc[b * R + c + 1] = y.y;
          }
        }
      } else {
        tc_fence_before();
        if (ARR == 0) { __syncwarp(); if (lane == 0) mbar_arrive_cluster(ready_lead + a * 8); }
        else { named_sync(1, 128 * NPW); if (threadIdx.x == 128) mbar_arrive_cluster(ready_lead + a * 8); }
      }
    }
#pragma unroll
    for (int c = 0; c < (WORK ? COLS : 1); ++c) keep += acc[c];
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = keep;
  tc_fence_before();
  __syncthreads();
  if (CG == 2) cluster_sync();
  if (warp == 2) { if (CG == 2) tmem_dealloc_cg2<512>(tb); else tmem_dealloc<512>(tb); }
}

static const uint8_t* g_src;
static unsigned long long* g_cyc2;
template <int CG, int N, int NACC, int WORK, int SPIN, int ARR, int NPW, int NOWAIT, int LOAD = 0>
void run(const char* name, float* dout, unsigned long long* dcyc) {
  auto k = k_loop<CG, N, NACC, WORK, SPIN, ARR, NPW, NOWAIT, LOAD>;
  const int smem = 1024 + 16384 + (N / CG) * 128 + 1024 + 4 * 8192;
  CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(148); cfg.blockDim = dim3(128 * (1 + NPW)); cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = CG; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
  cfg.attrs = at; cfg.numAttrs = 1;
  const int iters = 4000;
  CK(cudaLaunchKernelEx(&cfg, k, 64, dout, dcyc, g_src, g_cyc2));
  CK(cudaLaunchKernelEx(&cfg, k, iters, dout, dcyc, g_src, g_cyc2));
  CK(cudaDeviceSynchronize());
  unsigned long long h[148];
  CK(cudaMemcpy(h, dcyc, sizeof(h), cudaMemcpyDeviceToHost));
  double c = 0; int n = 0;
  for (int i = 0; i < 148; i += CG) { c += h[i]; ++n; }
  c /= n;
  const double mma = 2.0 * N;   // 4 x K=32 MMAs of 128 CG x N at 8192 MAC/clk/SM
  double l = 0;
  if (LOAD) {
    unsigned long long h2[148];
    CK(cudaMemcpy(h2, g_cyc2, sizeof(h2), cudaMemcpyDeviceToHost));
    for (int i = 0; i < 148; ++i) l += h2[i];
    l /= 148;
  }
  printf("  \"%s\": {\"clk_per_kblock\": %.1f, \"mma_floor_clk\": %.0f, \"load_B_per_clk_sm\": %.1f},\n", name,
         LOAD == 2 ? 0.0 : c / iters, mma, LOAD ? 3.0 * 8192 * iters / l : 0.0);
}

int main() {
  float* dout; unsigned long long* dcyc;
  CK(cudaMalloc(&dout, 4 * 148 * 1024)); CK(cudaMalloc(&dcyc, 8 * 148));
  uint8_t* src; CK(cudaMalloc(&src, 64 << 20)); CK(cudaMemset(src, 1, 64 << 20)); g_src = src;
  CK(cudaMalloc(&g_cyc2, 8 * 148));
  printf("{\n");
  // SPIN = issuer wait + 8 * promotion wait (0 production, 1 test_wait spin, 2 try_wait loop,
  // 3 try_wait 1 ms hint, 4 try_wait 20 us hint, 5 test_wait then try_wait)
  run<2, 256, 2, 1, 0, 0, 2, 0, 0>("work_w00", dout, dcyc);
  run<2, 256, 2, 1, 2 + 8 * 2, 0, 2, 0, 0>("work_w22", dout, dcyc);
  run<2, 256, 2, 1, 0 + 8 * 2, 0, 2, 0, 0>("work_w02", dout, dcyc);
  run<2, 256, 2, 1, 0 + 8 * 3, 0, 2, 0, 0>("work_w03", dout, dcyc);
  run<2, 256, 2, 1, 0 + 8 * 4, 0, 2, 0, 0>("work_w04", dout, dcyc);
  run<2, 256, 2, 1, 0 + 8 * 5, 0, 2, 0, 0>("work_w05", dout, dcyc);
  run<2, 256, 2, 1, 5 + 8 * 5, 0, 2, 0, 0>("work_w55", dout, dcyc);
  run<2, 256, 2, 1, 2 + 8 * 0, 0, 2, 0, 0>("work_w20", dout, dcyc);
  run<2, 256, 2, 0, 0, 0, 2, 0, 0>("nowork_w00", dout, dcyc);
  run<2, 256, 1, 1, 0, 0, 2, 0, 0>("nacc1_work_w00", dout, dcyc);
  run<2, 256, 1, 1, 2 + 8 * 2, 0, 2, 0, 0>("nacc1_work_w22", dout, dcyc);
  printf("  \"done\": 1\n}\n");
  return 0;
}
