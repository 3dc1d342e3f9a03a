// probe_ring.cu -- round-trip latency of the GEMM's accumulator ring on a CTA pair.
// One K-block = 4 pair MMAs (M=256, N=256, K=32 each, f8f6f4, operands in shared memory).
// Per iteration j the even CTA's issuer waits ready[j % R], issues the K-block into accumulator
// j % R (R = ring depth, 1 or 2), commits full[j % R] (multicast to both CTAs); in each CTA
// "promotion" warp 0 waits full, optionally loads its 32 lanes x 256 columns (tcgen05.ld), then
// arrives on the even CTA's ready barrier (remote from the odd CTA).  Reports clk per K-block:
//   mma_only   : back-to-back K-blocks, no ring (tensor-core rate)
//   ring R=1   : fully serialised: exec + commit->wake + arrive->wake + issue
//   ring R=2   : two accumulators (what the GEMM has at N=256)
// with and without the promotion's TMEM loads.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 probe_ring.cu -o probe_ring
#include <cuda_runtime.h>
#include <cstdio>
#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"
using namespace comet::sm100;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

constexpr int ITERS = 512;

template <int MODE, int R, int LOADS, int NPROMO = 1, int COLS = 256, int PB = 32, int MATH = 0>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(384, 1) k_ring(unsigned long long* out) {
  __shared__ __align__(8) uint64_t full[2], ready[2], done;
  __shared__ uint32_t tb_s;
  extern __shared__ __align__(1024) uint8_t tile[];    // A 16 KB + B 16 KB (contents irrelevant)
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const uint32_t rank = cluster_ctarank();
  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) { mbar_init(&full[i], 1); mbar_init(&ready[i], 2 * NPROMO); }
    mbar_init(&done, 1);
    fence_mbar_init();
  }
  if (w == 0) { tmem_alloc_cg2<512>(&tb_s); tmem_relinquish_cg2(); }
  tc_fence_before(); __syncthreads(); cluster_sync(); tc_fence_after();
  const uint32_t tb = tb_s;
  const uint32_t ready_lead = mapa_shared(smem_u32(&ready[0]), 0);
  const uint32_t sA = smem_u32(tile), sB = smem_u32(tile + 16384);
  const uint32_t id = idesc_f8f6f4_e4m3(256, 256);
  if (w == 1 && lane == 0 && rank == 0) {
    unsigned long long t0 = clock64();
    for (int j = 0; j < ITERS; ++j) {
      const int a = j % R;
      if (MODE == 1 && j >= R) mbar_wait(&ready[a], ((j / R) - 1) & 1);
      tc_fence_after();
      for (int k = 0; k < 4; ++k)
        mma_f8_ss_cg2(tb + a * 256, sdesc_kmajor_sw128(sA + 32 * k), sdesc_kmajor_sw128(sB + 32 * k), id, k);
      if (MODE == 1) tc_commit_mc(&full[a], 3);
    }
    tc_commit_mc(&done, 3);
    mbar_wait(&done, 0);
    out[0] = clock64() - t0;
  }
  if (MODE == 1 && w >= 4 && w < 4 + NPROMO) {   // promotion warps
    const int pw = w - 4;
    const uint32_t tcol = tb + ((uint32_t)(32 * (pw & 3)) << 16) + (pw >> 2) * COLS;
    float acc[MATH ? COLS : 1];
    for (int c = 0; c < (MATH ? COLS : 1); ++c) acc[c] = 0.f;
    const float2 s2 = make_float2(1.0001f, 1.0001f);
    for (int j = 0; j < ITERS; ++j) {
      const int a = j % R;
      mbar_wait(&full[a], (j / R) & 1);
      tc_fence_after();
      if (LOADS) {
        uint32_t vb[2][PB];
        uint32_t x = 0;
        tmem_ld_32x32b<PB>(tcol + a * 256, vb[0]);
        tmem_wait_ld();
#pragma unroll
        for (int b = 0; b < COLS / PB; ++b) {
          uint32_t* v = vb[b & 1];
          if (b + 1 < COLS / PB) tmem_ld_32x32b<PB>(tcol + a * 256 + (b + 1) * PB, vb[(b + 1) & 1]);
          if (MATH) {
#pragma unroll
            for (int c = 0; c < PB; c += 2) {
              float2 y = ffma2(make_float2(__uint_as_float(v[c]), __uint_as_float(v[c + 1])), s2,
                               make_float2(acc[b * PB + c], acc[b * PB + c + 1]));
              acc[b * PB + c] = y.x; acc[b * PB + c + 1] = y.y;
            }
          } else {
            x += v[0] ^ v[PB - 1];
          }
          if (b + 1 < COLS / PB) {
            tmem_wait_ld();
            if (b + 2 == COLS / PB) {
              tc_fence_before();
              __syncwarp();
              if (lane == 0 && j + R < ITERS) mbar_arrive_cluster(ready_lead + 8 * a);
            }
          }
        }
        if (x == 0x12345678u) out[15] = x;
        if (COLS / PB == 1) {
          tc_fence_before();
          __syncwarp();
          if (lane == 0 && j + R < ITERS) mbar_arrive_cluster(ready_lead + 8 * a);
        }
      } else {
        tc_fence_before();
        __syncwarp();
        if (lane == 0 && j + R < ITERS) mbar_arrive_cluster(ready_lead + 8 * a);
      }
    }
    if (MATH) {
      float t = 0.f;
      for (int c = 0; c < COLS; ++c) t += acc[c];
      if (t == 1.2345f) out[14] = 1;
    }
  }
  if (MODE == 1 && w != 4 && w != 1 && rank == 0 && threadIdx.x == 0) {
    // nothing: the done barrier is waited by the issuer
  }
  if (rank == 1 && w == 1 && lane == 0) mbar_wait(&done, 0);
  tc_fence_before();
  __syncthreads();
  cluster_sync();
  if (w == 0) tmem_dealloc_cg2<512>(tb);
}

template <int MODE, int R, int LOADS, int NPROMO = 1, int COLS = 256, int PB = 32, int MATH = 0>
double run(unsigned long long* d) {
  auto k = k_ring<MODE, R, LOADS, NPROMO, COLS, PB, MATH>;
  CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 32768));
  CK(cudaMemset(d, 0, 16 * 8));
  k<<<2, 384, 32768>>>(d);
  CK(cudaDeviceSynchronize());
  unsigned long long h;
  CK(cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost));
  return h / (double)ITERS;
}

int main() {
  unsigned long long* d;
  CK(cudaMalloc(&d, 16 * 8));
  run<0, 1, 0>(d);   // warm-up
  printf("{\"clk_per_kblock\": {\"mma_only\": %.1f, \"ring1\": %.1f, \"ring1_loads\": %.1f, "
         "\"ring2\": %.1f, \"ring2_loads\": %.1f, ",
         run<0, 1, 0>(d), run<1, 1, 0>(d), run<1, 1, 1>(d), run<1, 2, 0>(d), run<1, 2, 1>(d));
  printf("\"ring2_8w_128c_pb16_loads\": %.1f, \"ring2_8w_128c_pb16_math\": %.1f, "
         "\"ring2_8w_128c_pb32_math\": %.1f, \"ring2_4w_256c_pb16_math\": %.1f, \"ring2_8w_0loads\": %.1f}}\n",
         run<1, 2, 1, 8, 128, 16, 0>(d), run<1, 2, 1, 8, 128, 16, 1>(d), run<1, 2, 1, 8, 128, 32, 1>(d),
         run<1, 2, 1, 4, 256, 16, 1>(d), run<1, 2, 0, 8, 128, 16, 0>(d));
  return 0;
}
