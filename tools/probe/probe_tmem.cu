// probe_tmem.cu -- TMEM -> register load latency / throughput per shape, and FFMA2 issue rate.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 probe_tmem.cu -o probe_tmem
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>
#include <string>
#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"
using namespace comet::sm100;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__device__ __forceinline__ void ld32x32_x32(uint32_t a, uint32_t* r) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
    : "=r"(r[0]),"=r"(r[1]),"=r"(r[2]),"=r"(r[3]),"=r"(r[4]),"=r"(r[5]),"=r"(r[6]),"=r"(r[7]),"=r"(r[8]),"=r"(r[9]),"=r"(r[10]),"=r"(r[11]),"=r"(r[12]),"=r"(r[13]),"=r"(r[14]),"=r"(r[15]),"=r"(r[16]),"=r"(r[17]),"=r"(r[18]),"=r"(r[19]),"=r"(r[20]),"=r"(r[21]),"=r"(r[22]),"=r"(r[23]),"=r"(r[24]),"=r"(r[25]),"=r"(r[26]),"=r"(r[27]),"=r"(r[28]),"=r"(r[29]),"=r"(r[30]),"=r"(r[31]) : "r"(a));
}

// MODE 0: 32x32b.x32 (4 KB/warp), 1: 16x256b.x8 (4 KB/warp), 2: 2 x 16x256b.x8 in flight (8 KB),
// 3: 4 x 16x256b.x8 in flight (16 KB)
template <int MODE, int NW>
__global__ void __launch_bounds__(NW * 32, 1) k_tmem(int iters, uint32_t* out, unsigned long long* cyc) {
  __shared__ uint32_t tb_s;
  const int w = threadIdx.x / 32;
  if (w == 0) { tmem_alloc<512>(&tb_s); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t tb = tb_s;
  const uint32_t lane_base = (uint32_t)((w % 4) * 32) << 16;
  uint32_t x = 0;
  __syncthreads();
  unsigned long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
    const uint32_t col = (uint32_t)(((w / 4) * 64 + it * 32) & 255);
    uint32_t r[128];
    if (MODE == 0) { ld32x32_x32(tb + lane_base + col, r); }
    if (MODE >= 1) { tmem_ld_16x256b_x8(tb + lane_base + col, r); }
    if (MODE >= 2) { tmem_ld_16x256b_x8(tb + lane_base + (16 << 16) + col, r + 32); }
    if (MODE >= 3) { tmem_ld_16x256b_x8(tb + lane_base + col + 64, r + 64); tmem_ld_16x256b_x8(tb + lane_base + (16 << 16) + col + 64, r + 96); }
    tmem_wait_ld();
    constexpr int NR = MODE == 3 ? 128 : (MODE == 2 ? 64 : 32);
    // log-depth xor reduce
    x ^= r[0] ^ r[NR - 1] ^ r[NR / 2];
  }
  unsigned long long c1 = clock64();
  out[blockIdx.x * blockDim.x + threadIdx.x] = x;
  if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
  tc_fence_before(); __syncthreads();
  if (w == 0) tmem_dealloc<512>(tb);
}

// FFMA2 issue rate: NW warps, 8 independent chains of f32x2 per thread.
template <int NW>
__global__ void __launch_bounds__(NW * 32, 1) k_ffma2(int iters, float* out, unsigned long long* cyc) {
  float2 a[8];
  for (int j = 0; j < 8; ++j) a[j] = make_float2(threadIdx.x * 1e-3f + j, j * 0.5f);
  const float2 s = make_float2(0.999f, 1.001f);
  __syncthreads();
  unsigned long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 8; ++j) a[j] = ffma2(a[j], s, a[(j + 1) & 7]);
  }
  unsigned long long c1 = clock64();
  float t = 0; for (int j = 0; j < 8; ++j) t += a[j].x + a[j].y;
  out[blockIdx.x * blockDim.x + threadIdx.x] = t;
  if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
}

template <int MODE, int NW>
double run_tmem(int nsm, uint32_t* dout, unsigned long long* dcyc) {
  int iters = 4000;
  k_tmem<MODE, NW><<<nsm, NW * 32>>>(16, dout, dcyc);
  k_tmem<MODE, NW><<<nsm, NW * 32>>>(iters, dout, dcyc);
  CK(cudaDeviceSynchronize());
  std::vector<unsigned long long> h(nsm);
  CK(cudaMemcpy(h.data(), dcyc, nsm * 8, cudaMemcpyDeviceToHost));
  double c = 0; for (auto v : h) c += v; c /= nsm;
  double bytes_per_warp = MODE == 3 ? 16384 : (MODE == 2 ? 8192 : 4096);
  return NW * bytes_per_warp * iters / c;   // bytes / clk / SM
}

template <int NW>
double run_ffma2(int nsm, float* dout, unsigned long long* dcyc) {
  int iters = 8000;
  k_ffma2<NW><<<nsm, NW * 32>>>(16, dout, dcyc);
  k_ffma2<NW><<<nsm, NW * 32>>>(iters, dout, dcyc);
  CK(cudaDeviceSynchronize());
  std::vector<unsigned long long> h(nsm);
  CK(cudaMemcpy(h.data(), dcyc, nsm * 8, cudaMemcpyDeviceToHost));
  double c = 0; for (auto v : h) c += v; c /= nsm;
  return (double)NW * iters * 8 / c;   // FFMA2 warp-instructions per clk per SM
}

int main() {
  int nsm = 148;
  uint32_t* dout; unsigned long long* dcyc; float* fout;
  CK(cudaMalloc(&dout, 4 * nsm * 1024)); CK(cudaMalloc(&dcyc, 8 * nsm)); CK(cudaMalloc(&fout, 4 * nsm * 1024));
  printf("{\"tmem_ld_bytes_per_clk_sm\": {");
  printf("\"32x32b.x32_w4\": %.1f, ", run_tmem<0, 4>(nsm, dout, dcyc));
  printf("\"32x32b.x32_w8\": %.1f, ", run_tmem<0, 8>(nsm, dout, dcyc));
  printf("\"32x32b.x32_w16\": %.1f, ", run_tmem<0, 16>(nsm, dout, dcyc));
  printf("\"16x256b.x8_w4\": %.1f, ", run_tmem<1, 4>(nsm, dout, dcyc));
  printf("\"16x256b.x8_w8\": %.1f, ", run_tmem<1, 8>(nsm, dout, dcyc));
  printf("\"16x256b.x8x2_w4\": %.1f, ", run_tmem<2, 4>(nsm, dout, dcyc));
  printf("\"16x256b.x8x2_w8\": %.1f, ", run_tmem<2, 8>(nsm, dout, dcyc));
  printf("\"16x256b.x8x4_w4\": %.1f, ", run_tmem<3, 4>(nsm, dout, dcyc));
  printf("\"16x256b.x8x4_w8\": %.1f", run_tmem<3, 8>(nsm, dout, dcyc));
  printf("}, \"ffma2_warp_instr_per_clk_sm\": {");
  printf("\"w4\": %.2f, ", run_ffma2<4>(nsm, fout, dcyc));
  printf("\"w8\": %.2f, ", run_ffma2<8>(nsm, fout, dcyc));
  printf("\"w16\": %.2f}}\n", run_ffma2<16>(nsm, fout, dcyc));
  return 0;
}
