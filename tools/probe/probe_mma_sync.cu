// probe_mma_sync.cu -- checks the two register-level facts gemm_v.cu relies on, on the device:
// (1) the E4M3 -> s8 conversion of code bytes (cvt.rn.f16x2.e4m3x2 + 1536 bias + byte permute)
//     for every code of |q| <= 7, in every byte position;
// (2) the mma.sync m16n8k32 .s32.u8.s8 fragment layout (A rows g / g+8, k 4t.. / 16+4t..;
//     B k 4t.. / 16+4t.. of column g; C rows g / g+8, columns 2t, 2t+1) against a CPU product.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_mma_sync probe_mma_sync.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <cstdlib>

__device__ __forceinline__ uint32_t e4m3x4_to_s8(uint32_t e) {
  uint32_t h0, h1;
  asm("{\n\t.reg .b16 lo, hi;\n\tmov.b32 {lo, hi}, %2;\n\t"
      "cvt.rn.f16x2.e4m3x2 %0, lo;\n\tcvt.rn.f16x2.e4m3x2 %1, hi;\n\t}\n"
      : "=r"(h0), "=r"(h1) : "r"(e), "r"(e));
  const uint32_t bias = 0x66006600u;   // f16x2 {1536, 1536}: 1536 + q in [1024, 2048), ulp 1
  asm("add.rn.f16x2 %0, %0, %1;" : "+r"(h0) : "r"(bias));
  asm("add.rn.f16x2 %0, %0, %1;" : "+r"(h1) : "r"(bias));
  return __byte_perm(h0, h1, 0x6420);
}

__global__ void k_conv(const uint32_t* in, uint32_t* out, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = e4m3x4_to_s8(in[i]);
}

// A [16][32] u8 row-major, B [8][32] s8 (column n = token, k contiguous), D [16][8] s32
__global__ void k_mma(const uint8_t* A, const int8_t* B, int* D) {
  const int lane = threadIdx.x, g = lane >> 2, t = lane & 3;
  auto w4 = [](const void* p) { return *reinterpret_cast<const uint32_t*>(p); };
  const uint32_t a0 = w4(A + g * 32 + 4 * t), a1 = w4(A + (g + 8) * 32 + 4 * t);
  const uint32_t a2 = w4(A + g * 32 + 16 + 4 * t), a3 = w4(A + (g + 8) * 32 + 16 + 4 * t);
  const uint32_t b0 = w4(B + g * 32 + 4 * t), b1 = w4(B + g * 32 + 16 + 4 * t);
  int d[4] = {0, 0, 0, 0};
  asm volatile("mma.sync.aligned.m16n8k32.row.col.s32.u8.s8.s32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
               : "+r"(d[0]), "+r"(d[1]), "+r"(d[2]), "+r"(d[3])
               : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
  D[g * 8 + 2 * t] = d[0]; D[g * 8 + 2 * t + 1] = d[1];
  D[(g + 8) * 8 + 2 * t] = d[2]; D[(g + 8) * 8 + 2 * t + 1] = d[3];
}

int main() {
  // (1) conversion: E4M3 bytes of q = -7..7 in all byte positions
  const uint8_t e4[8] = {0x00, 0x38, 0x40, 0x44, 0x48, 0x4A, 0x4C, 0x4E};
  const int n = 15 * 15 * 4;
  uint32_t h_in[n], h_out[n];
  int8_t want[n][4];
  int idx = 0;
  for (int qa = -7; qa <= 7; ++qa)
    for (int qb = -7; qb <= 7; ++qb)
      for (int rot = 0; rot < 4; ++rot, ++idx) {
        int q[4] = {qa, qb, (qa + qb) / 2, -qa};
        uint32_t v = 0;
        for (int i = 0; i < 4; ++i) {
          const int qq = q[(i + rot) & 3];
          want[idx][i] = (int8_t)qq;
          const uint8_t b = e4[qq < 0 ? -qq : qq] | (qq < 0 ? 0x80 : 0);
          v |= (uint32_t)b << (8 * i);
        }
        h_in[idx] = v;
      }
  uint32_t *d_in, *d_out;
  cudaMalloc(&d_in, sizeof(h_in));
  cudaMalloc(&d_out, sizeof(h_out));
  cudaMemcpy(d_in, h_in, sizeof(h_in), cudaMemcpyHostToDevice);
  k_conv<<<(n + 255) / 256, 256>>>(d_in, d_out, n);
  cudaMemcpy(h_out, d_out, sizeof(h_out), cudaMemcpyDeviceToHost);
  int bad = 0;
  for (int i = 0; i < n; ++i)
    for (int j = 0; j < 4; ++j)
      if ((int8_t)(h_out[i] >> (8 * j)) != want[i][j]) {
        if (bad < 4) printf("conv mismatch word %08x byte %d: got %d want %d\n", h_in[i], j, (int8_t)(h_out[i] >> (8 * j)), want[i][j]);
        ++bad;
      }
  printf("{\"conversion_mismatches\": %d}\n", bad);
  // (2) fragment layout
  uint8_t hA[16 * 32];
  int8_t hB[8 * 32];
  int hD[16 * 8];
  srand(1);
  for (int i = 0; i < 16 * 32; ++i) hA[i] = (uint8_t)(rand() % 16);
  for (int i = 0; i < 8 * 32; ++i) hB[i] = (int8_t)(rand() % 255 - 127);
  uint8_t* dA; int8_t* dB; int* dD;
  cudaMalloc(&dA, sizeof(hA)); cudaMalloc(&dB, sizeof(hB)); cudaMalloc(&dD, sizeof(hD));
  cudaMemcpy(dA, hA, sizeof(hA), cudaMemcpyHostToDevice);
  cudaMemcpy(dB, hB, sizeof(hB), cudaMemcpyHostToDevice);
  k_mma<<<1, 32>>>(dA, dB, dD);
  cudaMemcpy(hD, dD, sizeof(hD), cudaMemcpyDeviceToHost);
  int badm = 0;
  for (int r = 0; r < 16; ++r)
    for (int c = 0; c < 8; ++c) {
      int s = 0;
      for (int k = 0; k < 32; ++k) s += (int)hA[r * 32 + k] * (int)hB[c * 32 + k];
      if (s != hD[r * 8 + c]) { if (badm < 4) printf("mma mismatch r %d c %d got %d want %d\n", r, c, hD[r * 8 + c], s); ++badm; }
    }
  printf("{\"mma_layout_mismatches\": %d}\n", badm);
  return (bad || badm) ? 1 : 0;
}
