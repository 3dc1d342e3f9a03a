// probe.cu -- B200 hardware probe for the W4Ax design decisions.
//
//  1. exactness + operand layout of tcgen05.mma kind::f8f6f4 (E4M3) and kind::i8, A from TMEM
//     ("TS") and from SMEM ("SS"):
//       f8:  A bytes 0x00..0x0F (offset-binary INT4 weight u = w+8, read as E4M3 = u * 2^-9,
//            subnormal for u < 8) x B = E4M3(x), x in [-7,7]  -> D must be the exact rational
//       i8:  random s8 x s8 and 16*w x s8                     -> D must be the exact integer
//  2. dense MMA throughput (MAC/clk/SM) for i8 / f8, TS / SS, N = 224 / 256
//  3. CUDA-core throughput of the promotion / widening instruction mix (lane-ops/clk/SM)
//  4. TMEM -> register load bandwidth (bytes/clk/SM)
// Prints one JSON object.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 probe.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <cmath>
#include <vector>
#include <random>
#include <string>

#include "../../paper_conf_asplos_liu0rxpwl0w25_b200/csrc/sm100.cuh"

using namespace comet::sm100;

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA error %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

// ------------------------------------------------------------------------------ 1. exactness
template <bool F8, bool TS>
__global__ void __launch_bounds__(128) k_mma_check(const uint8_t* A, const uint8_t* B, uint32_t* D, int N) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* sB = smem;               // 256 rows x 128 B
  uint8_t* sA = smem + 256 * 128;   // 128 rows x 128 B
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase_s;
  const int t = threadIdx.x, w = t / 32;
  for (int i = t; i < N * 8; i += 128) {
    int row = i / 8, ch = i % 8;
    *(uint4*)(sB + row * 128 + ((ch ^ (row & 7)) * 16)) = *(const uint4*)(B + row * 128 + ch * 16);
  }
  if (!TS) {
    for (int i = t; i < 128 * 8; i += 128) {
      int row = i / 8, ch = i % 8;
      *(uint4*)(sA + row * 128 + ((ch ^ (row & 7)) * 16)) = *(const uint4*)(A + row * 128 + ch * 16);
    }
  }
  if (w == 0) { tmem_alloc<512>(&tbase_s); tmem_relinquish(); }
  if (t == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tbase_s;
  const uint32_t lane_base = (uint32_t)(w * 32) << 16;
  if (TS) {
    uint32_t r[32];
    const uint32_t* row = (const uint32_t*)(A + t * 128);
#pragma unroll
    for (int j = 0; j < 32; ++j) r[j] = row[j];
    tmem_st32(tb + lane_base, r);
    tmem_wait_st();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (t == 0) {
    const uint32_t idesc = F8 ? idesc_f8f6f4_e4m3(128, N) : idesc_i8(128, N);
    for (int k = 0; k < 4; ++k) {
      uint64_t bd = sdesc_kmajor_sw128(smem_u32(sB) + 32 * k);
      if (TS) {
        if (F8) mma_f8_ts(tb + 64, tb + 8 * k, bd, idesc, k > 0);
        else    mma_i8_ts(tb + 64, tb + 8 * k, bd, idesc, k > 0);
      } else {
        uint64_t ad = sdesc_kmajor_sw128(smem_u32(sA) + 32 * k);
        if (F8) mma_f8_ss(tb + 64, ad, bd, idesc, k > 0);
        else    mma_i8_ss(tb + 64, ad, bd, idesc, k > 0);
      }
    }
    tc_commit(&bar);
  }
  __syncwarp();
  mbar_wait(&bar, 0);
  tc_fence_after();
  for (int c = 0; c < N; c += 16) {
    uint32_t r[16];
    tmem_ld16(tb + lane_base + 64 + c, r);
    tmem_wait_ld();
    for (int j = 0; j < 16; ++j) D[t * N + c + j] = r[j];
  }
  tc_fence_before();
  __syncthreads();
  if (w == 0) tmem_dealloc<512>(tb);
}

static double e4m3_to_double(uint8_t b) {
  int s = b >> 7, e = (b >> 3) & 15, m = b & 7;
  double v = (e == 0) ? std::ldexp((double)m, -9) : std::ldexp(1.0 + m / 8.0, e - 7);
  if (e == 15 && m == 7) v = NAN;
  return s ? -v : v;
}
static uint8_t e4m3_of_int(int x) {   // exact for |x| <= 16
  for (int b = 0; b < 256; ++b) if (e4m3_to_double((uint8_t)b) == (double)x && !(x == 0 && b != 0)) return (uint8_t)b;
  return 0xFF;
}

struct CheckResult { long mismatches; long total; double max_abs_err; };

template <bool F8, bool TS>
static CheckResult run_check(const std::vector<uint8_t>& A, const std::vector<uint8_t>& B, int N) {
  uint8_t *dA, *dB; uint32_t* dD;
  CK(cudaMalloc(&dA, 128 * 128)); CK(cudaMalloc(&dB, 256 * 128)); CK(cudaMalloc(&dD, 128 * 256 * 4));
  CK(cudaMemcpy(dA, A.data(), 128 * 128, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(dB, B.data(), N * 128, cudaMemcpyHostToDevice));
  size_t smem = 1024 + 256 * 128 + 128 * 128;
  CK(cudaFuncSetAttribute(k_mma_check<F8, TS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  k_mma_check<F8, TS><<<1, 128, smem>>>(dA, dB, dD, N);
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  std::vector<uint32_t> D(128 * N);
  CK(cudaMemcpy(D.data(), dD, 128 * N * 4, cudaMemcpyDeviceToHost));
  CheckResult r{0, 128L * N, 0.0};
  for (int m = 0; m < 128; ++m)
    for (int n = 0; n < N; ++n) {
      double ref = 0, got;
      for (int k = 0; k < 128; ++k) {
        if (F8) ref += e4m3_to_double(A[m * 128 + k]) * e4m3_to_double(B[n * 128 + k]);
        else ref += (double)(int8_t)A[m * 128 + k] * (double)(int8_t)B[n * 128 + k];
      }
      if (F8) { float f; memcpy(&f, &D[m * N + n], 4); got = f; }
      else got = (double)(int32_t)D[m * N + n];
      double err = fabs(got - ref);
      if (err != 0) r.mismatches++;
      if (err > r.max_abs_err) r.max_abs_err = err;
    }
  cudaFree(dA); cudaFree(dB); cudaFree(dD);
  return r;
}

// ------------------------------------------------------------------------------ 2. MMA peak
template <bool F8, bool TS, int N>
__global__ void __launch_bounds__(128, 1) k_mma_peak(int iters, unsigned long long* cyc) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase_s;
  const int t = threadIdx.x, w = t / 32;
  for (int i = t; i < (256 + 128) * 128 / 16; i += 128) ((uint4*)smem)[i] = make_uint4(0x01010101u * (i & 3), 0, 0, 0);
  if (w == 0) { tmem_alloc<512>(&tbase_s); tmem_relinquish(); }
  if (t == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
  fence_proxy_async_smem();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tbase_s;
  if (t == 0) {
    const uint32_t idesc = F8 ? idesc_f8f6f4_e4m3(128, N) : idesc_i8(128, N);
    const uint32_t sB = smem_u32(smem), sA = smem_u32(smem + 256 * 128);
    unsigned long long c0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        uint64_t bd = sdesc_kmajor_sw128(sB + 32 * k);
        if (TS) {
          if (F8) mma_f8_ts(tb + 256, tb + 8 * k, bd, idesc, 1);
          else    mma_i8_ts(tb + 256, tb + 8 * k, bd, idesc, 1);
        } else {
          uint64_t ad = sdesc_kmajor_sw128(sA + 32 * k);
          if (F8) mma_f8_ss(tb + 256, ad, bd, idesc, 1);
          else    mma_i8_ss(tb + 256, ad, bd, idesc, 1);
        }
      }
    }
    tc_commit(&bar);
    mbar_wait(&bar, 0);
    unsigned long long c1 = clock64();
    cyc[blockIdx.x] = c1 - c0;
  }
  tc_fence_before();
  __syncthreads();
  if (w == 0) tmem_dealloc<512>(tb);
}

// ------------------------------------------------------------------------------ 3. ALU mix
// op: 0 = I2FP (cvt.rn.f32.s32), 1 = FFMA, 2 = FFMA2 (f32x2), 3 = LOP3, 4 = FADD2, 5 = IADD3
template <int OP>
__global__ void __launch_bounds__(256) k_alu(int iters, float* out, unsigned long long* cyc) {
  float f[8]; int v[8];
  for (int j = 0; j < 8; ++j) { f[j] = threadIdx.x * 0.001f + j; v[j] = threadIdx.x + j * 7; }
  unsigned long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      if (OP == 0) { float g; asm volatile("cvt.rn.f32.s32 %0, %1;" : "=f"(g) : "r"(v[j])); v[j] ^= __float_as_int(g); }
      if (OP == 1) { asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(f[j]) : "f"(1.0001f), "f"(0.5f)); }
      if (OP == 2 && (j & 1) == 0) {
        float2 a = make_float2(f[j], f[j + 1]);
        a = ffma2(a, make_float2(1.0001f, 1.0002f), make_float2(0.5f, 0.25f));
        f[j] = a.x; f[j + 1] = a.y;
      }
      if (OP == 3) { asm volatile("lop3.b32 %0, %0, %1, %2, 0x6a;" : "+r"(v[j]) : "r"(0xF0F0F0F0), "r"(0x80808080)); }
      if (OP == 4 && (j & 1) == 0) {
        asm volatile("{\n\t.reg .b64 ra, rb;\n\tmov.b64 ra, {%0, %1};\n\tmov.b64 rb, {%2, %3};\n\t"
                     "add.rn.f32x2 ra, ra, rb;\n\tmov.b64 {%0, %1}, ra;\n\t}\n"
                     : "+f"(f[j]), "+f"(f[j + 1]) : "f"(0.5f), "f"(0.25f));
      }
      if (OP == 5) { asm volatile("add.s32 %0, %0, %1;" : "+r"(v[j]) : "r"(0x1234)); }
    }
  }
  unsigned long long c1 = clock64();
  float s = 0; for (int j = 0; j < 8; ++j) s += f[j] + v[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = c1 - c0;
}

// ------------------------------------------------------------------------------ 4. TMEM ld BW
template <int NWARPS>
__global__ void __launch_bounds__(NWARPS * 32, 1) k_tmem_ld(int iters, float* out, unsigned long long* cyc) {
  __shared__ uint32_t tbase_s;
  const int t = threadIdx.x, w = t / 32;
  if (w == 0) { tmem_alloc<512>(&tbase_s); tmem_relinquish(); }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tb = tbase_s;
  const uint32_t lane_base = (uint32_t)((w % 4) * 32) << 16;
  const uint32_t colbase = (w / 4) * 32;
  float acc = 0;
  unsigned long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
    uint32_t r[32];
    tmem_ld32(tb + lane_base + ((colbase + it * 64) & 511), r);
    tmem_wait_ld();
#pragma unroll
    for (int j = 0; j < 32; ++j) acc += __int_as_float(r[j]);
  }
  unsigned long long c1 = clock64();
  out[blockIdx.x * blockDim.x + t] = acc;
  if (t == 0) cyc[blockIdx.x] = c1 - c0;
  tc_fence_before();
  __syncthreads();
  if (w == 0) tmem_dealloc<512>(tb);
}

static double mean_cycles(unsigned long long* d, int n) {
  std::vector<unsigned long long> h(n);
  CK(cudaMemcpy(h.data(), d, n * 8, cudaMemcpyDeviceToHost));
  double s = 0; for (auto v : h) s += (double)v; return s / n;
}

template <bool F8, bool TS, int N>
static void run_peak(const char* name, int nsm, unsigned long long* dcyc, std::string& js) {
  size_t smem = 1024 + (256 + 128) * 128;
  CK(cudaFuncSetAttribute(k_mma_peak<F8, TS, N>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int iters = 4000;
  k_mma_peak<F8, TS, N><<<nsm, 128, smem>>>(100, dcyc);
  CK(cudaDeviceSynchronize());
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k_mma_peak<F8, TS, N><<<nsm, 128, smem>>>(iters, dcyc);
  cudaEventRecord(e1);
  CK(cudaEventSynchronize(e1));
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  double cyc = mean_cycles(dcyc, nsm);
  double macs_per_sm = (double)iters * 4 * 128.0 * N * 32;
  double mac_per_clk = macs_per_sm / cyc;
  double tops = 2.0 * macs_per_sm * nsm / (ms * 1e-3) / 1e12;
  char buf[256];
  snprintf(buf, sizeof buf, "\"%s\": {\"mac_per_clk_sm\": %.1f, \"tops\": %.1f, \"ms\": %.3f, \"mhz_eff\": %.0f}, ",
           name, mac_per_clk, tops, ms, cyc / (ms * 1e3));
  js += buf;
}

template <int OP>
static void run_alu(const char* name, int nsm, unsigned long long* dcyc, float* dout, std::string& js) {
  int blocks = nsm * 8, iters = 4096;
  k_alu<OP><<<blocks, 256>>>(64, dout, dcyc);
  CK(cudaDeviceSynchronize());
  k_alu<OP><<<blocks, 256>>>(iters, dout, dcyc);
  CK(cudaDeviceSynchronize());
  double cyc = mean_cycles(dcyc, blocks);
  // each SM runs 8 blocks concurrently (8*256 = 2048 threads)
  double lane_ops = (double)iters * 8 * 256 * 8;   // per SM (8 resident blocks)
  char buf[200];
  snprintf(buf, sizeof buf, "\"%s\": %.1f, ", name, lane_ops / cyc);
  js += buf;
}

int main() {
  cudaDeviceProp prop; CK(cudaGetDeviceProperties(&prop, 0));
  int nsm = prop.multiProcessorCount;
  std::string js = "{";
  char buf[512];
  snprintf(buf, sizeof buf, "\"gpu\": \"%s\", \"sms\": %d, \"l2_bytes\": %d, ", prop.name, nsm, prop.l2CacheSize);
  js += buf;

  std::mt19937 rng(1234);
  // --- exactness checks
  std::vector<uint8_t> A(128 * 128), B(256 * 128);
  uint8_t e4[15]; for (int x = -7; x <= 7; ++x) e4[x + 7] = e4m3_of_int(x);
  auto fill_f8 = [&](int mode) {
    for (int m = 0; m < 128; ++m) for (int k = 0; k < 128; ++k) {
      int u = rng() % 16;
      if (mode == 1) u = (m % 2) ? 15 : (k == 0 ? 15 : 1);
      if (mode == 2) u = (k % 32 == 0) ? 15 : (rng() % 2);
      A[m * 128 + k] = (uint8_t)u;                          // offset-binary nibble as E4M3 bits
    }
    for (int n = 0; n < 256; ++n) for (int k = 0; k < 128; ++k) {
      int x = (int)(rng() % 15) - 7;
      if (mode == 1) x = (n % 2) ? 7 : (k == 0 ? 7 : ((rng() & 1) ? 1 : -1));
      if (mode == 2) x = (k % 32 == 0) ? ((n & 1) ? 7 : -7) : (int)(rng() % 3) - 1;
      B[n * 128 + k] = e4[x + 7];
    }
  };
  struct Case { const char* name; int mode; int N; };
  for (int mode = 0; mode < 3; ++mode) {
    for (int N : {32, 224}) {
      fill_f8(mode);
      CheckResult r1 = run_check<true, true>(A, B, N);
      CheckResult r2 = run_check<true, false>(A, B, N);
      snprintf(buf, sizeof buf, "\"f8_mode%d_N%d\": {\"ts_mismatch\": %ld, \"ss_mismatch\": %ld, \"total\": %ld, \"ts_maxerr\": %g}, ",
               mode, N, r1.mismatches, r2.mismatches, r1.total, r1.max_abs_err);
      js += buf;
    }
  }
  for (int mode = 0; mode < 2; ++mode) {
    for (int m = 0; m < 128 * 128; ++m) A[m] = mode == 0 ? (uint8_t)(rng() & 255) : (uint8_t)(((rng() % 16) << 4));
    for (int m = 0; m < 256 * 128; ++m) { int x = (int)(rng() % 255) - 127; B[m] = (uint8_t)(int8_t)x; }
    CheckResult r1 = run_check<false, true>(A, B, 224);
    CheckResult r2 = run_check<false, false>(A, B, 224);
    snprintf(buf, sizeof buf, "\"i8_mode%d\": {\"ts_mismatch\": %ld, \"ss_mismatch\": %ld, \"total\": %ld}, ",
             mode, r1.mismatches, r2.mismatches, r1.total);
    js += buf;
  }
  // --- peaks
  unsigned long long* dcyc; float* dout;
  CK(cudaMalloc(&dcyc, 8 * nsm * 16)); CK(cudaMalloc(&dout, 4 * nsm * 8 * 256));
  run_peak<false, true, 256>("i8_ts_n256", nsm, dcyc, js);
  run_peak<false, true, 224>("i8_ts_n224", nsm, dcyc, js);
  run_peak<true, true, 256>("f8_ts_n256", nsm, dcyc, js);
  run_peak<true, true, 224>("f8_ts_n224", nsm, dcyc, js);
  run_peak<false, false, 256>("i8_ss_n256", nsm, dcyc, js);
  run_peak<true, false, 256>("f8_ss_n256", nsm, dcyc, js);
  run_peak<true, true, 128>("f8_ts_n128", nsm, dcyc, js);
  run_peak<true, true, 64>("f8_ts_n64", nsm, dcyc, js);
  run_peak<true, true, 32>("f8_ts_n32", nsm, dcyc, js);
  run_peak<true, true, 16>("f8_ts_n16", nsm, dcyc, js);
  // --- ALU
  js += "\"alu_lane_ops_per_clk_sm\": {";
  run_alu<0>("i2fp", nsm, dcyc, dout, js);
  run_alu<1>("ffma", nsm, dcyc, dout, js);
  run_alu<2>("ffma2", nsm, dcyc, dout, js);
  run_alu<3>("lop3", nsm, dcyc, dout, js);
  run_alu<4>("fadd2", nsm, dcyc, dout, js);
  run_alu<5>("iadd", nsm, dcyc, dout, js);
  js += "\"_\": 0}, ";
  // --- TMEM load bandwidth
  {
    int iters = 2000;
    k_tmem_ld<4><<<nsm, 128>>>(iters, dout, dcyc); CK(cudaDeviceSynchronize());
    double c4 = mean_cycles(dcyc, nsm);
    k_tmem_ld<8><<<nsm, 256>>>(iters, dout, dcyc); CK(cudaDeviceSynchronize());
    double c8 = mean_cycles(dcyc, nsm);
    k_tmem_ld<16><<<nsm, 512>>>(iters, dout, dcyc); CK(cudaDeviceSynchronize());
    double c16 = mean_cycles(dcyc, nsm);
    snprintf(buf, sizeof buf, "\"tmem_ld_bytes_per_clk_sm\": {\"w4\": %.1f, \"w8\": %.1f, \"w16\": %.1f}, ",
             4.0 * 32 * 32 * 4 * iters / c4, 8.0 * 32 * 32 * 4 * iters / c8, 16.0 * 32 * 32 * 4 * iters / c16);
    js += buf;
  }
  js += "\"ok\": true}";
  printf("%s\n", js.c_str());
  return 0;
}
