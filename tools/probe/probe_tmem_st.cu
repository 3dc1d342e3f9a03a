// probe_tmem_st.cu -- register -> TMEM store throughput per shape and wait batching (the decode
// kernel's widen warps store 2 x 32x32b.x32 per stage and wait).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 probe_tmem_st.cu -o probe_tmem_st
#include <cuda_runtime.h>
#include <cstdio>
#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"
using namespace comet::sm100;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__device__ __forceinline__ void st16x256_x8(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.16x256b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,"
      "%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
      "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]),
      "r"(r[16]), "r"(r[17]), "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]),
      "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]),
      "r"(r[30]), "r"(r[31])
      : "memory");
}

// MODE 0: 32x32b.x32 (4 KB / warp / store), 1: 16x256b.x8 (4 KB); PER = stores between waits
template <int MODE, int NW, int PER>
__global__ void __launch_bounds__(NW * 32, 1) k_st(int iters, unsigned long long* cyc) {
  __shared__ uint32_t tb_s;
  const int w = threadIdx.x / 32;
  if (w == 0) { tmem_alloc<512>(&tb_s); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tb = tb_s;
  const uint32_t lane_base = (uint32_t)((w % 4) * 32) << 16;
  uint32_t r[32];
  for (int i = 0; i < 32; ++i) r[i] = threadIdx.x * 33 + i;
  __syncthreads();
  unsigned long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int p = 0; p < PER; ++p) {
      const uint32_t col = (uint32_t)((((w / 4) * 128) + ((it * PER + p) * 32)) & 511);
      if (MODE == 0) tmem_st32(tb + lane_base + col, r);
      else st16x256_x8(tb + lane_base + col, r);
    }
    tmem_wait_st();
    r[0] += 1;
  }
  unsigned long long c1 = clock64();
  if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
  tc_fence_before(); __syncthreads();
  if (w == 0) tmem_dealloc<512>(tb);
}

template <int MODE, int NW, int PER>
void run(const char* name) {
  unsigned long long* d; CK(cudaMalloc(&d, 148 * 8));
  const int iters = 2000;
  k_st<MODE, NW, PER><<<148, NW * 32>>>(10, d);
  CK(cudaDeviceSynchronize());
  k_st<MODE, NW, PER><<<148, NW * 32>>>(iters, d);
  CK(cudaDeviceSynchronize());
  unsigned long long h[148]; CK(cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost));
  double c = 0; for (int i = 0; i < 148; ++i) c += h[i]; c /= 148;
  const double bytes = (double)iters * PER * NW * 4096.0;
  printf("{\"shape\": \"%s\", \"warps\": %d, \"stores_per_wait\": %d, \"clk_per_iter\": %.1f, \"B_per_clk_per_SM\": %.1f}\n",
         name, NW, PER, c / iters, bytes / c);
  CK(cudaFree(d));
}

int main() {
  run<0, 4, 1>("32x32b.x32"); run<0, 4, 2>("32x32b.x32"); run<0, 4, 4>("32x32b.x32");
  run<0, 8, 1>("32x32b.x32"); run<0, 8, 2>("32x32b.x32"); run<0, 8, 4>("32x32b.x32");
  run<0, 16, 2>("32x32b.x32");
  run<1, 4, 2>("16x256b.x8"); run<1, 8, 2>("16x256b.x8"); run<1, 8, 4>("16x256b.x8");
  return 0;
}
