// probe_smem.cu -- does tcgen05.mma (SS operands) share shared-memory bandwidth with LSU
// traffic (LDS/STS)?  Warp 0 issues back-to-back SS MMAs (M=128, N=256, K=32, f8f6f4) while
// warps 4..11 stream LDS.128 + STS.128 over a separate region.  Reports MMA MAC/clk/SM and LSU
// bytes/clk/SM alone and together.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 probe_smem.cu -o probe_smem
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"
using namespace comet::sm100;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

// DO_MMA / DO_LSU select the activities.  LSU_MODE 0: LDS.128+STS.128 pairs, 1: STS only, 2: LDS only
template <bool DO_MMA, bool DO_LSU, int LSU_MODE, int NMMA_N>
__global__ void __launch_bounds__(384, 1) k(int mma_iters, int lsu_iters, unsigned long long* out) {
  extern __shared__ uint8_t raw[];
  uint8_t* smem = raw + ((1024u - (smem_u32(raw) & 1023u)) & 1023u);
  __shared__ uint64_t bar;
  __shared__ uint32_t tb_s;
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (w == 0) { tmem_alloc<512>(&tb_s); tmem_relinquish(); }
  if (threadIdx.x == 32) { mbar_init(&bar, 1); fence_mbar_init(); }
  for (int i = threadIdx.x; i < 200 * 1024 / 16; i += 384) ((uint4*)smem)[i] = make_uint4(0x01010101u * (i & 7), 0, 0, 0);
  fence_proxy_async_smem();
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tb = tb_s;
  unsigned long long t0 = clock64(), t1 = t0;
  if (w == 1 && lane == 0 && DO_MMA) {
    const uint32_t sA = smem_u32(smem), sB = smem_u32(smem + 16384);
    const uint32_t id = idesc_f8f6f4_e4m3(128, NMMA_N);
    for (int it = 0; it < mma_iters; ++it)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk)
        mma_f8_ss(tb, sdesc_kmajor_sw128(sA + 32 * kk), sdesc_kmajor_sw128(sB + 32 * kk), id, 1);
    tc_commit(&bar);
    mbar_wait(&bar, 0);
    t1 = clock64();
    out[blockIdx.x * 4 + 0] = t1 - t0;
  }
  if (w >= 4 && DO_LSU) {
    const uint32_t base = smem_u32(smem + 64 * 1024) + (w - 4) * 16384 + lane * 16;
    uint4 acc = make_uint4(0, 0, 0, 0);
    for (int it = 0; it < lsu_iters; ++it) {
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint32_t a = base + ((it * 8 + j) & 31) * 512;
        if (LSU_MODE != 1) {
          uint4 v = lds128(a);
          acc.x ^= v.x; acc.y += v.y;
        }
        if (LSU_MODE != 2) {
          asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a ^ 256u), "r"(acc.x), "r"(acc.y), "r"(it), "r"(j));
        }
      }
    }
    t1 = clock64();
    if (lane == 0) atomicMax(&out[blockIdx.x * 4 + 1], t1 - t0);
    if (acc.x == 12345 && acc.y == 777) out[blockIdx.x * 4 + 3] = 1;
  }
  tc_fence_before(); __syncthreads();
  if (w == 0) tmem_dealloc<512>(tb);
}

template <bool M, bool L, int LM, int NN>
void run(const char* name, int mma_iters, int lsu_iters) {
  int nsm = 148;
  unsigned long long* d;
  CK(cudaMalloc(&d, nsm * 4 * 8));
  CK(cudaMemset(d, 0, nsm * 4 * 8));
  int smem = 210 * 1024;
  CK(cudaFuncSetAttribute(k<M, L, LM, NN>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  k<M, L, LM, NN><<<nsm, 384, smem>>>(mma_iters / 10, lsu_iters / 10, d);
  CK(cudaMemset(d, 0, nsm * 4 * 8));
  k<M, L, LM, NN><<<nsm, 384, smem>>>(mma_iters, lsu_iters, d);
  CK(cudaDeviceSynchronize());
  std::vector<unsigned long long> h(nsm * 4);
  CK(cudaMemcpy(h.data(), d, nsm * 32, cudaMemcpyDeviceToHost));
  double cm = 0, cl = 0;
  for (int i = 0; i < nsm; ++i) { cm += h[i * 4]; cl += h[i * 4 + 1]; }
  cm /= nsm; cl /= nsm;
  double mac = M ? (double)mma_iters * 4 * 128.0 * NN * 32 / cm : 0;
  double lsu_bytes = (double)lsu_iters * 8 * 8 * 32 * 16 * (LM == 0 ? 2 : 1);
  double bpc = L ? lsu_bytes / cl : 0;
  printf("\"%s\": {\"mma_mac_per_clk\": %.0f, \"lsu_bytes_per_clk\": %.1f, \"mma_cyc\": %.0f, \"lsu_cyc\": %.0f}, ", name, mac, bpc, cm, cl);
  cudaFree(d);
}

int main() {
  printf("{");
  run<true, false, 0, 256>("mma_only_n256", 4000, 0);
  run<false, true, 0, 256>("lsu_only_ldsts", 0, 4000);
  run<true, true, 0, 256>("mma_plus_ldsts", 4000, 4000);
  run<false, true, 1, 256>("lsu_only_sts", 0, 4000);
  run<true, true, 1, 256>("mma_plus_sts", 4000, 4000);
  run<false, true, 2, 256>("lsu_only_lds", 0, 4000);
  run<true, true, 2, 256>("mma_plus_lds", 4000, 4000);
  run<true, false, 0, 128>("mma_only_n128", 4000, 0);
  run<true, true, 0, 128>("mma128_plus_ldsts", 4000, 4000);
  printf("\"ok\": 1}\n");
  return 0;
}
