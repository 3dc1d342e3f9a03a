// probe_ldg.cu -- HBM streaming rate of plain LDG.128 weight reads on B200 (the ceiling of a
// CUDA-core / mma.sync decode GEMM), timed like bench.py's decode sweep: back-to-back launches
// cycling over weight copies > 2 x L2, mean per launch.
//   mode 0: grid-stride contiguous uint4 loads, U loads in flight per thread
//   mode 1: GEMV pattern -- a warp owns 16 rows [N][K/2] and walks K in 128-channel blocks
//           (lane (g, t): 16 B of row g and of row g + 8 per block), U blocks in flight;
//           rows split over the grid in contiguous row ranges
//   mode 2 / 3: CTA-level (128-row group, K-block) units on the row-major / tiled layout (k_units)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_ldg probe_ldg.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

__device__ __forceinline__ uint4 ldg_stream(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

template <int U>
__global__ void k_stream(const uint4* __restrict__ p, size_t n, uint32_t* sink) {
  uint32_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + (U - 1) * stride < n; i += U * stride) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ldg_stream(p + i + u * stride);
#pragma unroll
    for (int u = 0; u < U; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  for (; i < n; i += stride) { uint4 v = ldg_stream(p + i); acc ^= v.x ^ v.y ^ v.z ^ v.w; }
  if (acc == 0x12345678u) sink[0] = acc;
}

// rows of rowbytes bytes; warp w handles 16-row tiles; tiles split over warps contiguously
template <int U>
__global__ void k_gemv(const uint8_t* __restrict__ w, int N, int rowbytes, uint32_t* sink) {
  const int lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int gw = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, nw = (gridDim.x * blockDim.x) >> 5;
  const int tiles = N / 16;
  const int nblk = rowbytes / 64;
  uint32_t acc = 0;
  // contiguous (tile, block) work range per warp
  const long long units = (long long)tiles * nblk;
  const long long u0 = units * gw / nw, u1 = units * (gw + 1) / nw;
  for (long long u = u0; u < u1; u += U) {
    uint4 v[U][2];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      const long long uu = u + k < u1 ? u + k : u1 - 1;
      const int tile = (int)(uu / nblk), b = (int)(uu % nblk);
      const uint8_t* r0 = w + ((size_t)(tile * 16 + g) * rowbytes) + b * 64 + t * 16;
      v[k][0] = ldg_stream(r0);
      v[k][1] = ldg_stream(r0 + (size_t)8 * rowbytes);
    }
#pragma unroll
    for (int k = 0; k < U; ++k) acc ^= v[k][0].x ^ v[k][1].y ^ v[k][0].z ^ v[k][1].w;
  }
  if (acc == 0x12345678u) sink[0] = acc;
}

// CTA-level (128-row group, K-block) units as gemm_v.cu walks them; warp w reads rows 16 w ..
// 16 w + 15 of the unit (lane (g, t): 16 B of row g and of row g + 8).  BLOCKED = 0: the
// row-major [N][K/2] layout (rows 4 KB apart); BLOCKED = 1: a tiled layout
// [N/128][K/128][128 rows][64 B] in which a unit is one contiguous 8 KB tile and a CTA's range
// is contiguous memory.
template <int U, int BLOCKED>
__global__ void k_units(const uint8_t* __restrict__ w, int N, int rowbytes, uint32_t* sink) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int nb = rowbytes / 64;
  const long long units = (long long)(N / 128) * nb;
  const long long u0 = units * blockIdx.x / gridDim.x, u1 = units * (blockIdx.x + 1) / gridDim.x;
  uint32_t acc = 0;
  for (long long u = u0; u < u1; u += U) {
    uint4 v[U][2];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      const long long uu = u + k < u1 ? u + k : u1 - 1;
      const long long grp = uu / nb;
      const int b = (int)(uu - grp * nb);
      const uint8_t* r0;
      size_t off8;
      if (BLOCKED) { r0 = w + (size_t)uu * 8192 + (warp * 16 + g) * 64 + t * 16; off8 = 512; }
      else { r0 = w + (size_t)(grp * 128 + warp * 16 + g) * rowbytes + b * 64 + t * 16; off8 = (size_t)8 * rowbytes; }
      v[k][0] = ldg_stream(r0);
      v[k][1] = ldg_stream(r0 + off8);
    }
#pragma unroll
    for (int k = 0; k < U; ++k) acc ^= v[k][0].x ^ v[k][1].y ^ v[k][0].z ^ v[k][1].w;
  }
  if (acc == 0x12345678u) sink[0] = acc;
}

int main(int argc, char** argv) {
  int dev = 0, nsm = 0;
  CK(cudaSetDevice(dev));
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  uint32_t* sink;
  CK(cudaMalloc(&sink, 4));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  const int rowbytes = 4096;
  for (int N : {28672, 10240}) {
    const size_t bytes = (size_t)N * rowbytes;
    const int ncopy = (int)((300ull << 20) / bytes) + 2;
    std::vector<uint8_t*> bufs(ncopy);
    for (auto& b : bufs) { CK(cudaMalloc(&b, bytes)); CK(cudaMemset(b, 1, bytes)); }
    for (int mode = 0; mode < 4; ++mode) {
      for (int ctas : {1, 2, 4, 8}) {
        for (int U : {2, 4, 8}) {
          if (mode >= 2 && ctas == 1) continue;
          auto launch = [&](int i) {
            const int grid = nsm * ctas;
            if (mode == 0) {
              const size_t n = bytes / 16;
              if (U == 2) k_stream<2><<<grid, 256>>>((const uint4*)bufs[i % ncopy], n, sink);
              else if (U == 4) k_stream<4><<<grid, 256>>>((const uint4*)bufs[i % ncopy], n, sink);
              else k_stream<8><<<grid, 256>>>((const uint4*)bufs[i % ncopy], n, sink);
            } else if (mode == 2 || mode == 3) {
              const bool bl = mode == 3;
              if (U == 2) (bl ? k_units<2, 1> : k_units<2, 0>)<<<grid, 256>>>(bufs[i % ncopy], N, rowbytes, sink);
              else if (U == 4) (bl ? k_units<4, 1> : k_units<4, 0>)<<<grid, 256>>>(bufs[i % ncopy], N, rowbytes, sink);
              else (bl ? k_units<8, 1> : k_units<8, 0>)<<<grid, 256>>>(bufs[i % ncopy], N, rowbytes, sink);
            } else {
              if (U == 2) k_gemv<2><<<grid, 256>>>(bufs[i % ncopy], N, rowbytes, sink);
              else if (U == 4) k_gemv<4><<<grid, 256>>>(bufs[i % ncopy], N, rowbytes, sink);
              else k_gemv<8><<<grid, 256>>>(bufs[i % ncopy], N, rowbytes, sink);
            }
          };
          for (int i = 0; i < 2 * ncopy; ++i) launch(i);
          CK(cudaEventRecord(e0));
          const int iters = 10 * ncopy;
          for (int i = 0; i < iters; ++i) launch(i);
          CK(cudaEventRecord(e1));
          CK(cudaEventSynchronize(e1));
          float ms = 0;
          CK(cudaEventElapsedTime(&ms, e0, e1));
          const double us = ms * 1e3 / iters;
          printf("{\"N\": %d, \"MB\": %.1f, \"mode\": %d, \"ctas_per_sm\": %d, \"U\": %d, \"us\": %.2f, \"GBps\": %.1f}\n",
                 N, bytes / 1e6, mode, ctas, U, us, bytes / us / 1e3);
        }
      }
    }
    for (auto& b : bufs) CK(cudaFree(b));
  }
  return 0;
}
