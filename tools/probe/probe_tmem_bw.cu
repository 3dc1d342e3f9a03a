// probe_tmem_bw.cu -- TMEM -> register read bandwidth per SM as a function of warps and loads in
// flight per warp (32x32b.x32 loads, NLD of them issued before one tcgen05.wait::ld), with and
// without a concurrent MMA stream writing another TMEM region (the prefill promotion's situation:
// each K-block of 128 products per output needs one 4-byte accumulator read, 256 B/clk/SM at the
// full kind::f8f6f4 / kind::i8 MMA rate).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 probe_tmem_bw.cu -o probe_tmem_bw
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"
using namespace comet::sm100;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

template <int NW, int NLD, int MMA>
__global__ void __launch_bounds__(NW * 32 + 32, 1) k_bw(int iters, uint32_t* out, unsigned long long* cyc) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  __shared__ uint32_t holder;
  __shared__ uint64_t bar;
  __shared__ volatile int stop;
  const int w = threadIdx.x / 32;
  for (int i = threadIdx.x; i < 32768; i += blockDim.x) smem[i] = (uint8_t)(i * 7);
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); stop = 0; }
  if (w == 0) { tmem_alloc<512>(&holder); tmem_relinquish(); }
  fence_proxy_async_smem();
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tb = holder;
  uint32_t x = 0;
  if (w == NW) {               // MMA stream into columns 256..511 (N = 256, M = 128, kind::i8)
    if (MMA) {
      const uint32_t id = idesc_i8(128, 256);
      int n = 0;
      while (!stop) {
        if (elect_one()) {
#pragma unroll
          for (int k = 0; k < 4; ++k)
            mma_i8_ss(tb + 256, sdesc_kmajor_sw128(smem_u32(smem) + 32 * k), sdesc_kmajor_sw128(smem_u32(smem) + 32 * k), id, k);
          tc_commit(&bar);
        }
        __syncwarp();
        mbar_wait(&bar, (uint32_t)(n & 1));
        ++n;
      }
    }
  } else {
    const uint32_t lane_base = (uint32_t)((w % 4) * 32) << 16;
    unsigned long long c0 = clock64();
    for (int it = 0; it < iters; ++it) {
      uint32_t r[32 * NLD];
#pragma unroll
      for (int l = 0; l < NLD; ++l) {
        const uint32_t col = (uint32_t)(((w / 4) * 32 * NLD + l * 32 + it * 8) & 255);
        tmem_ld_32x32b<32>(tb + lane_base + col, r + 32 * l);
      }
      tmem_wait_ld();
#pragma unroll
      for (int i = 0; i < 32 * NLD; i += 8) x ^= r[i];
    }
    unsigned long long c1 = clock64();
    if (threadIdx.x == 0) { cyc[blockIdx.x] = c1 - c0; stop = 1; }
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
  tc_fence_before(); __syncthreads(); tc_fence_after();
  if (w == 0) tmem_dealloc<512>(tb);
}

template <int NW, int NLD, int MMA>
void run(uint32_t* dout, unsigned long long* dcyc) {
  auto k = k_bw<NW, NLD, MMA>;
  CK(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 33 * 1024));
  const int iters = 4000;
  k<<<148, NW * 32 + 32, 33 * 1024>>>(16, dout, dcyc);
  k<<<148, NW * 32 + 32, 33 * 1024>>>(iters, dout, dcyc);
  CK(cudaDeviceSynchronize());
  unsigned long long h[148];
  CK(cudaMemcpy(h, dcyc, sizeof(h), cudaMemcpyDeviceToHost));
  double c = 0; for (int i = 0; i < 148; ++i) c += h[i]; c /= 148;
  printf("  \"w%d_ld%d_mma%d\": %.1f,\n", NW, NLD, MMA, (double)NW * NLD * 4096.0 * iters / c);
}

int main() {
  uint32_t* dout; unsigned long long* dcyc;
  CK(cudaMalloc(&dout, 4 * 148 * 1024)); CK(cudaMalloc(&dcyc, 8 * 148));
  printf("{\"tmem_read_B_per_clk_sm\": {\n");
  run<4, 1, 0>(dout, dcyc); run<4, 2, 0>(dout, dcyc); run<4, 4, 0>(dout, dcyc);
  run<8, 1, 0>(dout, dcyc); run<8, 2, 0>(dout, dcyc); run<8, 4, 0>(dout, dcyc);
  run<16, 1, 0>(dout, dcyc); run<16, 2, 0>(dout, dcyc);
  run<8, 2, 1>(dout, dcyc); run<8, 4, 1>(dout, dcyc); run<16, 2, 1>(dout, dcyc);
  printf("  \"done\": 1}}\n");
  return 0;
}
