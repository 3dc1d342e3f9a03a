// probe_sync.cu -- issue cost (clk per op, one thread, back to back) of the synchronisation
// primitives on the GEMM's per-K-block path: mbarrier arrive (local / remote in a CTA pair),
// try_wait on an already-completed phase, tcgen05.commit (cta_group::1, and ::2 multicast),
// tcgen05.fence::before/after_thread_sync, and a 4-MMA K-block issue.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 probe_sync.cu -o probe_sync
#include <cuda_runtime.h>
#include <cstdio>
#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"
using namespace comet::sm100;
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

constexpr int N_OPS = 256;

__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(128, 1) k_sync(unsigned long long* out) {
  __shared__ __align__(8) uint64_t bars[N_OPS + 8];
  __shared__ uint32_t tb_s;
  __shared__ __align__(1024) uint8_t tile[32768];
  const int w = threadIdx.x / 32, lane = threadIdx.x % 32;
  const uint32_t rank = cluster_ctarank();
  if (threadIdx.x == 0) {
    for (int i = 0; i < N_OPS + 8; ++i) mbar_init(&bars[i], (1 << 20) - 1);
    fence_mbar_init();
  }
  if (w == 0) { tmem_alloc_cg2<512>(&tb_s); tmem_relinquish_cg2(); }
  tc_fence_before(); __syncthreads(); cluster_sync(); tc_fence_after();
  const uint32_t tb = tb_s;
  unsigned long long r[12] = {0};
  if (threadIdx.x == 0 && rank == 0) {
    unsigned long long t0, t1;
    // 1. local arrive
    t0 = clock64();
    for (int i = 0; i < N_OPS; ++i) mbar_arrive(&bars[i]);
    t1 = clock64(); r[0] = t1 - t0;
    // 2. remote arrive (peer CTA)
    const uint32_t peer = mapa_shared(smem_u32(&bars[0]), 1);
    t0 = clock64();
    for (int i = 0; i < N_OPS; ++i) mbar_arrive_cluster(peer + 8 * i);
    t1 = clock64(); r[1] = t1 - t0;
    // 3. try_wait on completed phase: init a barrier with count 1 and complete it
    mbar_init(&bars[N_OPS], 1); fence_mbar_init(); mbar_arrive(&bars[N_OPS]);
    t0 = clock64();
    for (int i = 0; i < N_OPS; ++i) mbar_wait(&bars[N_OPS], 0);
    t1 = clock64(); r[2] = t1 - t0;
    // 4. tcgen05 fences
    t0 = clock64();
    for (int i = 0; i < N_OPS; ++i) tc_fence_after();
    t1 = clock64(); r[3] = t1 - t0;
    t0 = clock64();
    for (int i = 0; i < N_OPS; ++i) tc_fence_before();
    t1 = clock64(); r[4] = t1 - t0;
    // 5. commit, cta_group::2 multicast (no MMA outstanding)
    t0 = clock64();
    for (int i = 0; i < N_OPS; ++i) tc_commit_mc(&bars[i], 3);
    t1 = clock64(); r[5] = t1 - t0;
    // 6. K-block of 4 pair MMAs (M=256, N=256) + 1 multicast commit, back to back
    const uint32_t sA = smem_u32(tile), sB = smem_u32(tile + 16384);
    const uint32_t id = idesc_f8f6f4_e4m3(256, 256);
    t0 = clock64();
    for (int i = 0; i < 64; ++i) {
      for (int k = 0; k < 4; ++k) mma_f8_ss_cg2(tb, sdesc_kmajor_sw128(sA + 32 * k), sdesc_kmajor_sw128(sB + 32 * k), id, 1);
      tc_commit_mc(&bars[i], 3);
    }
    t1 = clock64(); r[6] = t1 - t0;
    // 7. K-block of 4 pair MMAs + 3 commits
    t0 = clock64();
    for (int i = 0; i < 64; ++i) {
      for (int k = 0; k < 4; ++k) mma_f8_ss_cg2(tb, sdesc_kmajor_sw128(sA + 32 * k), sdesc_kmajor_sw128(sB + 32 * k), id, 1);
      tc_commit_mc(&bars[i], 3); tc_commit_mc(&bars[i + 64], 3); tc_commit_mc(&bars[i + 128], 3);
    }
    t1 = clock64(); r[7] = t1 - t0;
    // 8. K-block of 4 MMAs, no commit
    t0 = clock64();
    for (int i = 0; i < 64; ++i)
      for (int k = 0; k < 4; ++k) mma_f8_ss_cg2(tb, sdesc_kmajor_sw128(sA + 32 * k), sdesc_kmajor_sw128(sB + 32 * k), id, 1);
    t1 = clock64(); r[8] = t1 - t0;
    // drain
    mbar_init(&bars[N_OPS + 1], 1); fence_mbar_init();
    tc_commit_mc(&bars[N_OPS + 1], 1);
    mbar_wait(&bars[N_OPS + 1], 0);
    // 9. syncwarp-free elect + arrive pattern: arrive from 32 lanes? (lane 0 only here)
    for (int i = 0; i < 9; ++i) out[i] = r[i];
  }
  __syncthreads();
  cluster_sync();
  if (w == 0) tmem_dealloc_cg2<512>(tb);
}

int main() {
  unsigned long long* d;
  CK(cudaMalloc(&d, 16 * 8));
  CK(cudaMemset(d, 0, 16 * 8));
  k_sync<<<2, 128>>>(d);
  CK(cudaDeviceSynchronize());
  unsigned long long h[16];
  CK(cudaMemcpy(h, d, 16 * 8, cudaMemcpyDeviceToHost));
  printf("{\"clk_per_op\": {\"arrive_local\": %.1f, \"arrive_remote\": %.1f, \"try_wait_done\": %.1f, "
         "\"fence_after\": %.1f, \"fence_before\": %.1f, \"commit_cg2_mc\": %.1f}, "
         "\"clk_per_kblock\": {\"4mma_1commit\": %.1f, \"4mma_3commit\": %.1f, \"4mma_nocommit\": %.1f}}\n",
         h[0] / (double)N_OPS, h[1] / (double)N_OPS, h[2] / (double)N_OPS, h[3] / (double)N_OPS,
         h[4] / (double)N_OPS, h[5] / (double)N_OPS, h[6] / 64.0, h[7] / 64.0, h[8] / 64.0);
  return 0;
}
