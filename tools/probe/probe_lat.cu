// probe_lat.cu -- latencies on the promotion warp's per-K-block chain (one CTA per SM, all SMs):
//  (1) tcgen05.ld 32x32b.x16 / .x32 issue -> wait::ld round trip, one warp, tensor core idle;
//  (2) the same while another warp streams cta_group::1 MMAs (M=128, N=256) into other columns;
//  (3) mbarrier try_wait vs test_wait on an already-completed phase.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 probe_lat.cu -o probe_lat
#include <cuda_runtime.h>
#include <cstdio>
#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"
using namespace comet::sm100;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

constexpr int ITERS = 256;

__device__ __forceinline__ bool test_wait(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred P;\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 P, [%1], %2;\n\t"
      "selp.b32 %0, 1, 0, P;\n\t}\n"
      : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
  return ok != 0;
}

template <int MMA_BG>
__global__ void __launch_bounds__(128, 1) k_lat(unsigned long long* out, uint32_t* sink) {
  __shared__ __align__(8) uint64_t bars[4];
  __shared__ uint32_t tb_s;
  __shared__ volatile int stop;
  extern __shared__ __align__(1024) uint8_t tile[];    // 48 KB operands for the MMA stream
  const int w = threadIdx.x / 32;
  if (threadIdx.x == 0) {
    mbar_init(&bars[0], 1); mbar_init(&bars[1], 1); mbar_init(&bars[2], 1); fence_mbar_init();
    stop = 0;
  }
  if (w == 0) { tmem_alloc<512>(&tb_s); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tb = tb_s;
  if (w == 1 && MMA_BG) {
    if (threadIdx.x == 32) {
      const uint32_t sA = smem_u32(tile), sB = smem_u32(tile + 16384);
      const uint32_t id = idesc_f8f6f4_e4m3(128, 256);
      int n = 0;
      while (!stop && n < 100000) {
        for (int k = 0; k < 4; ++k) mma_f8_ss(tb + 256, sdesc_kmajor_sw128(sA + 32 * k), sdesc_kmajor_sw128(sB + 32 * k), id, 1);
        ++n;
        if ((n & 7) == 0) {   // bound the queue: wait for the MMAs issued so far
          tc_commit(&bars[1]);
          mbar_wait(&bars[1], ((n >> 3) - 1) & 1);
        }
      }
      tc_commit(&bars[2]);          // drain before dealloc
      mbar_wait(&bars[2], 0);
    }
  }
  if (w == 0) {
    uint32_t r[32];
    uint32_t acc = 0;
    // warm-up
    tmem_ld_32x32b_x16(tb, r); tmem_wait_ld();
    unsigned long long t0 = clock64();
    for (int i = 0; i < ITERS; ++i) {
      tmem_ld_32x32b_x16(tb + (i & 7) * 16, r);
      tmem_wait_ld();
      acc += r[0] ^ r[15];
    }
    unsigned long long t1 = clock64();
    for (int i = 0; i < ITERS; ++i) {
      tmem_ld_32x32b_x32(tb + (i & 3) * 32, r);
      tmem_wait_ld();
      acc += r[0] ^ r[31];
    }
    unsigned long long t2 = clock64();
    // two x16 loads per wait
    for (int i = 0; i < ITERS; ++i) {
      tmem_ld_32x32b_x16(tb + (i & 3) * 32, r);
      tmem_ld_32x32b_x16(tb + (i & 3) * 32 + 16, r + 16);
      tmem_wait_ld();
      acc += r[0] ^ r[31];
    }
    unsigned long long t3 = clock64();
    if (threadIdx.x == 0) {
      // completed phase: arrive once, then wait on parity 0 repeatedly
      mbar_arrive(&bars[0]);
      unsigned long long a0 = clock64();
      for (int i = 0; i < ITERS; ++i) mbar_wait(&bars[0], 0);
      unsigned long long a1 = clock64();
      uint32_t ok = 0;
      for (int i = 0; i < ITERS; ++i) ok += test_wait(smem_u32(&bars[0]), 0);
      unsigned long long a2 = clock64();
      if (blockIdx.x == 0) {
        out[MMA_BG * 8 + 0] = (t1 - t0);
        out[MMA_BG * 8 + 1] = (t2 - t1);
        out[MMA_BG * 8 + 2] = (t3 - t2);
        out[MMA_BG * 8 + 3] = (a1 - a0);
        out[MMA_BG * 8 + 4] = (a2 - a1);
        out[MMA_BG * 8 + 5] = ok;
      }
      stop = 1;
    }
    sink[blockIdx.x * 128 + threadIdx.x] = acc;
  }
  tc_fence_before();
  __syncthreads();
  if (w == 0) tmem_dealloc<512>(tb);
}

int main() {
  unsigned long long* d;
  uint32_t* sink;
  CK(cudaMalloc(&d, 16 * 8));
  CK(cudaMemset(d, 0, 16 * 8));
  CK(cudaMalloc(&sink, 148 * 128 * 4));
  CK(cudaFuncSetAttribute(k_lat<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 49152));
  CK(cudaFuncSetAttribute(k_lat<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 49152));
  k_lat<0><<<148, 128, 49152>>>(d, sink);
  CK(cudaDeviceSynchronize());
  k_lat<1><<<148, 128, 49152>>>(d, sink);
  CK(cudaDeviceSynchronize());
  unsigned long long h[16];
  CK(cudaMemcpy(h, d, 16 * 8, cudaMemcpyDeviceToHost));
  for (int m = 0; m < 2; ++m)
    printf("{\"mma_background\": %d, \"clk\": {\"ld_x16_wait\": %.1f, \"ld_x32_wait\": %.1f, \"ld_2x16_wait\": %.1f, "
           "\"try_wait_done\": %.1f, \"test_wait_done\": %.1f}, \"test_ok\": %llu}\n",
           m, h[m * 8] / (double)ITERS, h[m * 8 + 1] / (double)ITERS, h[m * 8 + 2] / (double)ITERS,
           h[m * 8 + 3] / (double)ITERS, h[m * 8 + 4] / (double)ITERS, h[m * 8 + 5]);
  return 0;
}
