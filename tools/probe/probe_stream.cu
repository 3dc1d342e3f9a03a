// probe_stream.cu -- HBM streaming rate of the decode GEMM's weight-read pattern on B200.
//
// A persistent kernel (one CTA per SM) streams a packed weight matrix [N][K/2] bytes
// (LLaMA-3-70B gate/up: N = 28672, K/2 = 4096 B) through a TMA -> mbarrier ring with no compute:
// one producer thread, one consumer warp that only releases the slot.  Units = (128-row tile,
// K-chunk of `inner` bytes), tile-major, split into contiguous ranges per CTA (as stream-K).
//   mode 0: 2D tensor map over the row-major matrix, box = inner bytes x `rows` rows
//   mode 1: blocked layout ([N/rows][K/2/inner][rows][inner], each unit contiguous), 1D bulk copy
//   mode 2: 2D tensor map, but each CTA walks units K-chunk-major inside a 4-tile band
// L2 is flushed (a 256 MiB write) before every timed launch.  Prints one JSON line per config.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>

#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"

using namespace comet::sm100;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

struct Prm {
  CUtensorMap map;
  CUtensorMap map4;   // 64-row boxes (mode 4)
  const uint8_t* base;
  long long units, units_per_tile;
  int unit_bytes, inner, rows, stages, mode;
  long long l2_tiles;
};

// Reads a buffer (clean L2 lines replace the dirty ones the memset left behind).
__global__ void k_read(const uint4* p, size_t n, uint32_t* sink) {
  uint32_t acc = 0;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
    uint4 v = p[i];
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x12345678u) *sink = acc;
}

__global__ void __launch_bounds__(384) k_stream(const __grid_constant__ Prm P) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  __shared__ uint64_t full[32], empty[32];
  const int S = P.stages;
  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    fence_mbar_init();
  }
  __syncthreads();
  const long long u0 = P.units * blockIdx.x / gridDim.x, u1 = P.units * (blockIdx.x + 1) / gridDim.x;
  if (P.mode >= 5) {
    // NP independent producer/consumer warp pairs (warps 2p / 2p+1), stages split between them.
    // mode 5: L2-resident 32 MB window; mode 6: the whole matrix streamed from HBM
    const int NP = blockDim.x / 64;
    const int pair = threadIdx.x / 64, role = (threadIdx.x / 32) & 1;
    if ((threadIdx.x & 31) != 0) return;
    const int S2 = S / NP;
    int st = 0; uint32_t ph = 0;
    for (long long u = u0 + pair; u < u1; u += NP) {
      const int sidx = pair * S2 + st;
      if (role == 0) {
        mbar_wait(&empty[sidx], ph ^ 1);
        mbar_arrive_expect_tx(&full[sidx], P.unit_bytes);
        const long long t = P.mode == 5 ? (u + (long long)blockIdx.x * 7) % (P.l2_tiles) : u;
        tma_load_2d(smem + sidx * P.unit_bytes, &P.map, &full[sidx], (int)((t % P.units_per_tile) * P.inner), (int)((t / P.units_per_tile) * P.rows));
      } else {
        mbar_wait(&full[sidx], ph);
        mbar_arrive(&empty[sidx]);
      }
      if (++st == S2) { st = 0; ph ^= 1; }
    }
    return;
  }
  if (threadIdx.x == 0) {
    int st = 0; uint32_t ph = 0;
    for (long long u = u0; u < u1; ++u) {
      mbar_wait(&empty[st], ph ^ 1);
      mbar_arrive_expect_tx(&full[st], P.unit_bytes);
      const long long tile = u / P.units_per_tile, kc = u % P.units_per_tile;
      if (P.mode == 3 || P.mode == 4) {
        // mode 4: the unit is split into `rows/64` boxes of 64 rows (several TMA ops per stage)
        const long long t = (u + (long long)blockIdx.x * 7) % (P.l2_tiles);
        const int c0 = (int)((t % P.units_per_tile) * P.inner), r0 = (int)((t / P.units_per_tile) * P.rows);
        if (P.mode == 3) {
          tma_load_2d(smem + st * P.unit_bytes, &P.map, &full[st], c0, r0);
        } else {
          for (int b = 0; b < P.rows / 64; ++b)
            tma_load_2d(smem + st * P.unit_bytes + b * 64 * P.inner, &P.map4, &full[st], c0, r0 + 64 * b);
        }
      } else if (P.mode == 1) {
        bulk_load(smem + st * P.unit_bytes, P.base + u * P.unit_bytes, P.unit_bytes, &full[st]);
      } else {
        tma_load_2d(smem + st * P.unit_bytes, &P.map, &full[st], (int)(kc * P.inner), (int)(tile * P.rows));
      }
      if (++st == S) { st = 0; ph ^= 1; }
    }
  } else if (threadIdx.x == 32) {
    int st = 0; uint32_t ph = 0;
    for (long long u = u0; u < u1; ++u) {
      mbar_wait(&full[st], ph);
      mbar_arrive(&empty[st]);
      if (++st == S) { st = 0; ph ^= 1; }
    }
  }
}

int main(int argc, char** argv) {
  const long long N = 28672, KB = 4096;   // rows, bytes per row
  const size_t bytes = (size_t)N * KB;
  uint8_t* d; CK(cudaMalloc(&d, bytes)); CK(cudaMemset(d, 0x5A, bytes));
  uint8_t* fl; CK(cudaMalloc(&fl, 256 << 20));
  uint8_t* fl2; CK(cudaMalloc(&fl2, 256 << 20)); CK(cudaMemset(fl2, 1, 256 << 20));
  uint32_t* sink; CK(cudaMalloc(&sink, 4));
  const int flush_mode = argc > 1 ? atoi(argv[1]) : 1;
  int nsm = 0; CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
  cudaDriverEntryPointQueryResult q; void* fnp = nullptr;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fnp, cudaEnableDefault, &q));
  auto enc = (PFN_cuTensorMapEncodeTiled_v12000)fnp;
  CK(cudaFuncSetAttribute(k_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  printf("{\"flush_mode\": %d}\n", flush_mode);
  for (int mult : {4, 8, 16}) {   // reference: plain 128-bit loads over the same matrix
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    std::vector<float> ts;
    for (int it = 0; it < 12; ++it) {
      CK(cudaMemsetAsync(fl, it, 256 << 20));
      if (flush_mode) k_read<<<nsm * 8, 256>>>((const uint4*)fl2, (256 << 20) / 16, sink);
      cudaEventRecord(a);
      k_read<<<nsm * mult, 256>>>((const uint4*)d, bytes / 16, sink);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      float ms; cudaEventElapsedTime(&ms, a, b);
      if (it >= 2) ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    const float ms = ts[ts.size() / 2];
    printf("{\"ldg_read_ctas_per_sm\": %d, \"us\": %.2f, \"GBps\": %.1f}\n", mult, ms * 1e3, bytes / (ms * 1e-3) / 1e9);
  }
  struct C { int mode, inner, rows, stages, l2, ctas_per_sm, np = 1; };
  std::vector<C> cfgs = {
      {0, 64, 128, 8, 2, 1}, {0, 64, 128, 16, 2, 1}, {0, 64, 128, 24, 2, 1}, {0, 64, 128, 16, 0, 1},
      {0, 128, 128, 8, 2, 1}, {0, 128, 128, 12, 2, 1}, {0, 256, 64, 12, 2, 1}, {0, 256, 128, 6, 2, 1},
      {1, 64, 128, 8, 0, 1}, {1, 64, 128, 16, 0, 1}, {1, 64, 128, 24, 0, 1}, {1, 128, 128, 12, 0, 1},
      {0, 64, 128, 12, 2, 2}, {1, 64, 128, 12, 0, 2}, {1, 64, 128, 12, 0, 3}, {1, 128, 128, 8, 0, 2},
      {1, 256, 128, 4, 0, 2}, {1, 256, 128, 6, 0, 1}, {1, 512, 128, 3, 0, 1},
      {3, 128, 128, 4, 2, 1}, {3, 128, 128, 8, 2, 1}, {3, 128, 128, 12, 2, 1}, {3, 64, 128, 16, 2, 1},
      {3, 128, 128, 6, 2, 2}, {3, 128, 64, 16, 2, 1}, {3, 128, 256, 4, 2, 1},
      {4, 128, 128, 8, 2, 1}, {4, 128, 256, 4, 2, 1}, {5, 128, 128, 8, 2, 1, 2}, {5, 128, 128, 12, 2, 1, 2}, {5, 128, 128, 8, 2, 1, 4}, {5, 128, 128, 12, 2, 1, 4},
      {6, 128, 128, 8, 2, 1, 2}, {6, 128, 128, 12, 2, 1, 4}, {6, 128, 128, 8, 2, 1, 4}, {6, 64, 128, 16, 2, 1, 4}, {6, 128, 128, 12, 2, 1, 6},
  };
  for (auto c : cfgs) {
    Prm P{};
    P.base = d; P.inner = c.inner; P.rows = c.rows; P.stages = c.stages; P.mode = c.mode;
    P.unit_bytes = c.inner * c.rows;
    P.units_per_tile = KB / c.inner;
    P.units = (N / c.rows) * P.units_per_tile;
    P.l2_tiles = (32ll << 20) / P.unit_bytes;      // mode 3: a 32 MB L2-resident window
    if (c.mode >= 3 && c.mode != 6) P.units *= 4;                 // stream 4x the matrix size from L2
    if (P.unit_bytes * c.stages > 200 * 1024 / c.ctas_per_sm || c.stages > 32) continue;
    cuuint64_t dims[2] = {(cuuint64_t)KB, (cuuint64_t)N};
    cuuint64_t str[1] = {(cuuint64_t)KB};
    cuuint32_t box[2] = {(cuuint32_t)std::min(c.inner, 256), (cuuint32_t)c.rows};
    cuuint32_t es[2] = {1, 1};
    CUtensorMapL2promotion pr = c.l2 == 2 ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B
                               : (c.l2 == 1 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B : CU_TENSOR_MAP_L2_PROMOTION_NONE);
    if (enc(&P.map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_NONE, pr, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
      printf("{\"error\": \"encode\", \"inner\": %d}\n", c.inner);
      continue;
    }
    {
      cuuint32_t box4[2] = {(cuuint32_t)std::min(c.inner, 256), 64u};
      enc(&P.map4, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, d, dims, str, box4, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_NONE, pr, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    }
    const int grid = nsm * c.ctas_per_sm;
    const int smem = P.unit_bytes * c.stages + 1024;
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    std::vector<float> ts;
    for (int it = 0; it < 12; ++it) {
      CK(cudaMemsetAsync(fl, it, 256 << 20));
      if (flush_mode) k_read<<<nsm * 8, 256>>>((const uint4*)fl2, (256 << 20) / 16, sink);
      cudaEventRecord(a);
      k_stream<<<grid, c.mode >= 5 ? 64 * c.np : 64, smem>>>(P);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      float ms; cudaEventElapsedTime(&ms, a, b);
      if (it >= 2) ts.push_back(ms);
    }
    CK(cudaGetLastError());
    std::sort(ts.begin(), ts.end());
    const float ms = ts[ts.size() / 2];
    const double tot = (double)P.units * P.unit_bytes;
    printf("{\"mode\": %d, \"np\": %d, \"inner\": %d, \"rows\": %d, \"stages\": %d, \"l2promo\": %d, \"ctas_per_sm\": %d, "
           "\"us\": %.2f, \"GBps\": %.1f}\n", c.mode, c.np, c.inner, c.rows, c.stages, c.l2, c.ctas_per_sm,
           ms * 1e3, tot / (ms * 1e-3) / 1e9);
  }
  return 0;
}
