// gemm.cu -- the W4Ax GEMM on sm_100a (kernel 2), persistent and warp-specialised.
//
//   Y[m, n] = s_w[n] * sum_b s_a[m,b] * acc_b[m,n]
//
// One CTA per SM walks the planner's work list (tile, K-block range).  An output
// tile is 128 weight rows (n) x NT tokens (m).  The MMA runs "transposed": the weight tile is
// the A operand (M = 128 rows, held in TENSOR MEMORY after widening), the activation tile is
// the B operand (N = NT tokens, TMA-staged in shared memory, 128-byte swizzle), so the tokens
// become the MMA N dimension and decode-sized M still fills an instruction.
//
// Roles (512 threads, 16 warps):
//   warp 0      TMA producer: activation tile [NT x 128 B], packed weight tile [128 x 64 B]
//               and the block's scales s_a[b][m0 .. m0+NT) into a STAGES-deep mbarrier ring.
//   warp 1      MMA issuer (one thread): per K-block 4 x tcgen05.mma (K = 32) into a fresh
//               TMEM accumulator; INT4 blocks use kind::f8f6f4 (E4M3), INT8 blocks kind::i8.
//   warp 2      TMEM allocator.
//   warps 4-7   widen: packed INT4 weight row -> 128 bytes in 3 instructions per 8 values
//               (the B200 form of the paper's location switch + zero extension),
//               tcgen05.st into one of two TMEM A buffers.  INT4 block: byte = u = w+8, read by
//               the FP8 tensor core as u * 2^-9 exactly.  INT8 block: byte = 16*w (s8).
//   warps 8-15  promotion ("dequant"): per K-block, tcgen05.ld the accumulator and fold
//               it into FP32 registers with the block's per-token scale (one FFMA2 per two
//               elements for INT4 blocks, the accumulator is already FP32); at the end of the
//               tile the FP32 result is scaled by s_w and stored (or, for a tile split across
//               CTAs, exchanged through the stream-K workspace).
//
// Exactness: INT4 block: acc = 2^-9 * sum_k x_k (w_k + 8) with every term an integer multiple
// of 2^-9 and |sum| < 2^14 -> exact in FP32 (checked bit-exactly against the oracle through the
// debug accumulators); the +8 offset is removed with corr[m] = 8 sum_b s_a qsum (kernel 1).
// INT8 block: acc = 16 * sum_k x_k w_k exactly in INT32.
#include <algorithm>
#include <cstdlib>
#include "gemm_common.cuh"

namespace comet {
namespace gemm {
namespace {
constexpr uint32_t kAcol = 0;        // TMEM columns [0, 64): two widened-weight A buffers
constexpr uint32_t kAccCol = 64;     // TMEM columns [64, 64 + 2 NT): two accumulators

template <int NT>
struct Cfg {
  static constexpr int ACTIVE_WGS = NT >= 32 ? 2 : 1;          // promotion warpgroups in use
  static constexpr int COLS = NT / ACTIVE_WGS;                 // accumulator columns per WG
  static constexpr int NACC = (64 + 3 * NT <= 512) ? 3 : 2;    // accumulator buffers in TMEM
  static constexpr int X_BYTES = NT * 128;
  static constexpr int W_BYTES = kTileW * 64;
  static constexpr int STAGE_BYTES = X_BYTES + W_BYTES;
  static constexpr int STAGES_RAW = (196 * 1024) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_RAW > 10 ? 10 : STAGES_RAW;
  static constexpr int SMEM_DATA = STAGES * STAGE_BYTES + kSRing * NT * 4;
  static constexpr int N_BARS = 2 * STAGES + 4 + 2 * NACC + 2 * kSRing;
  static constexpr int SMEM_BYTES = 1024 + SMEM_DATA + N_BARS * 8 + 16 + kMaxBlocks;
  static_assert(COLS % 16 == 0, "promotion chunks of 16 columns");
  static_assert(NACC * NT + 64 <= 512, "TMEM budget");
};

template <int NT, int DEBUG>
__global__ void __launch_bounds__(kThreads, 1) k_w4ax(const __grid_constant__ GemmParams P) {
  using C = Cfg<NT>;
  constexpr int S = C::STAGES;
  constexpr int NACC = C::NACC;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // keep the pointer derived from the __shared__ array (shared address space) when aligning
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sX = smem;
  uint8_t* sW = sX + S * C::X_BYTES;
  float* sS = reinterpret_cast<float*>(sW + S * C::W_BYTES);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::SMEM_DATA);
  uint64_t* full = bars;                    // [S]    TMA -> (MMA, widen)
  uint64_t* empty = bars + S;               // [S]    (MMA commit + 4 widen warps) -> TMA
  uint64_t* a_full = bars + 2 * S;          // [2]    widen -> MMA
  uint64_t* a_empty = a_full + 2;           // [2]    MMA commit -> widen
  uint64_t* acc_full = a_full + 4;          // [NACC] MMA commit -> promotion
  uint64_t* acc_empty = acc_full + NACC;    // [NACC] promotion -> MMA
  uint64_t* s_full = acc_empty + NACC;      // [kSRing] TMA -> promotion
  uint64_t* s_empty = s_full + kSRing;      // [kSRing] promotion -> TMA
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + C::N_BARS);
  uint8_t* s_tags = reinterpret_cast<uint8_t*>(tmem_holder + 4);
  const uint32_t s_tags_a = smem_u32(s_tags);
  const uint32_t sW_a = smem_u32(sW);
  const uint32_t sS_a = smem_u32(sS);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const bool debug = DEBUG != 0;
  const int it_begin = debug ? (int)blockIdx.x : P.cta_begin[blockIdx.x];
  const int it_end = debug ? (int)blockIdx.x + 1 : P.cta_begin[blockIdx.x + 1];
  const int nb = P.nb;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&P.map_x);
    tma_prefetch(&P.map_w);
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1 + 4);
    }
    for (int i = 0; i < 2; ++i) {
      mbar_init(&a_full[i], 4);
      mbar_init(&a_empty[i], 1);
    }
    for (int i = 0; i < NACC; ++i) {
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_empty[i], 4 * C::ACTIVE_WGS);
    }
    for (int i = 0; i < kSRing; ++i) {
      mbar_init(&s_full[i], 1);
      mbar_init(&s_empty[i], 4 * C::ACTIVE_WGS);
    }
    fence_mbar_init();
  }
  if (warp == 2) {
    tmem_alloc<512>(tmem_holder);
    tmem_relinquish();
  }
  for (int i = threadIdx.x; i < nb; i += kThreads) s_tags[i] = P.tags.get(i) ? 1 : 0;
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_holder;

  if (warp < 4) {
    setmaxnreg_dec<40>();
    if (warp == 0 && lane == 0) {
      // ------------------------------------------------------------------ TMA producer
      int stage = 0, ss = 0;
      uint32_t ph = 0, sph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = load_item(P, it, debug);
        const int n_tile = w.tile / P.n_m_tiles, m_tile = w.tile % P.n_m_tiles;
        const int m0 = m_tile * NT, n0 = n_tile * kTileW;
        const int64_t srows = min((int64_t)NT, P.Mp - m0);
        const uint32_t sbytes = (uint32_t)(srows * 4);
        for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
          mbar_wait(&empty[stage], ph ^ 1);
          mbar_arrive_expect_tx(&full[stage], C::STAGE_BYTES);
          tma_load_2d(sX + stage * C::X_BYTES, &P.map_x, &full[stage], kb * 128, m0);
          tma_load_2d(sW + stage * C::W_BYTES, &P.map_w, &full[stage], kb * 64, n0);
          mbar_wait(&s_empty[ss], sph ^ 1);
          mbar_arrive_expect_tx(&s_full[ss], sbytes);
          bulk_load(sS + ss * NT, P.scales + (int64_t)kb * P.Mp + m0, sbytes, &s_full[ss]);
          if (++stage == S) { stage = 0; ph ^= 1; }
          if (++ss == kSRing) { ss = 0; sph ^= 1; }
        }
      }
    } else if (warp == 1 && lane == 0) {
      // ------------------------------------------------------------------ MMA issuer
      const uint32_t id_f8 = idesc_f8f6f4_e4m3(128, NT);
      const uint32_t id_i8 = idesc_i8(128, NT);
      int stage = 0, ab = 0, accb = 0;
      uint32_t ph = 0, aph = 0, accph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = load_item(P, it, debug);
        for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
          mbar_wait(&acc_empty[accb], accph ^ 1);
          mbar_wait(&full[stage], ph);
          mbar_wait(&a_full[ab], aph);
          tc_fence_after();
          const uint32_t d = tbase + kAccCol + accb * NT;
          const uint32_t a = tbase + kAcol + ab * 32;
          const uint32_t sx = smem_u32(sX + stage * C::X_BYTES);
          if (lds_u8(s_tags_a + kb)) {
#pragma unroll
            for (int k = 0; k < 4; ++k) mma_i8_ts(d, a + 8 * k, sdesc_kmajor_sw128(sx + 32 * k), id_i8, k);
          } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) mma_f8_ts(d, a + 8 * k, sdesc_kmajor_sw128(sx + 32 * k), id_f8, k);
          }
          tc_commit(&empty[stage]);
          tc_commit(&a_empty[ab]);
          tc_commit(&acc_full[accb]);
          if (++stage == S) { stage = 0; ph ^= 1; }
          if (++ab == 2) { ab = 0; aph ^= 1; }
          if (++accb == NACC) { accb = 0; accph ^= 1; }
        }
      }
    }
  } else if (warp < 8) {
    setmaxnreg_dec<80>();
    // -------------------------------------------------------------------- widen (W -> TMEM A)
    const int q = warp & 3;
    const int r = q * 32 + lane;                  // TMEM lane = weight row within the tile
    const uint32_t lane_addr = (uint32_t)(q * 32) << 16;
    const int sw = (r >> 1) & 3;                  // TMA 64-byte swizzle: chunk ^= row bits [1:2]
    int stage = 0, ab = 0;
    uint32_t ph = 0, aph = 0;
    for (int it = it_begin; it < it_end; ++it) {
      const WorkItem w = load_item(P, it, debug);
      for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
        const bool is8 = lds_u8(s_tags_a + kb) != 0;
        mbar_wait(&full[stage], ph);
        const uint32_t wt = sW_a + stage * C::W_BYTES + r * 64;
        uint4 c[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) c[j] = lds128(wt + ((j ^ sw) << 4));
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[stage]);
        uint32_t o[32];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const uint32_t pw[4] = {c[j].x, c[j].y, c[j].z, c[j].w};
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            const uint32_t p = pw[i];
            const int g = j * 4 + i;
            if (is8) {
              o[2 * g] = ((p << 4) & 0xF0F0F0F0u) ^ 0x80808080u;
              o[2 * g + 1] = (p & 0xF0F0F0F0u) ^ 0x80808080u;
            } else {
              o[2 * g] = p & 0x0F0F0F0Fu;
              o[2 * g + 1] = (p >> 4) & 0x0F0F0F0Fu;
            }
          }
        }
        mbar_wait(&a_empty[ab], aph ^ 1);
        tc_fence_after();
        tmem_st32(tbase + kAcol + ab * 32 + lane_addr, o);
        tmem_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&a_full[ab]);
        if (++stage == S) { stage = 0; ph ^= 1; }
        if (++ab == 2) { ab = 0; aph ^= 1; }
      }
    }
  } else {
    setmaxnreg_inc<192>();
    // -------------------------------------------------------------------- promotion + epilogue
    // TMEM accumulator: lane = weight row (n), column = token (m).  With the 16x256b load shape
    // thread t of warp quarter q owns lanes 32q + 16h + t/4 + 8i (h, i in {0,1}) and columns
    // col0 + 8j + 2(t%4) + e (j < NJ, e in {0,1}): only NJ*2 distinct tokens, so the block's
    // per-token scales for this thread are NJ float2 loads issued before the accumulator wait.
    const int pw = warp - 8;
    const int wg = pw >> 2;
    const int q = warp & 3;
    const int t0 = lane & 3, t1 = lane >> 2;
    const int col0 = wg * C::COLS;
    constexpr int NJ = C::COLS / 8;                 // 8-column groups per WG
    constexpr int NB1 = NJ > 8 ? 8 : NJ;            // repetitions in the first load batch
    constexpr int NB2 = NJ - NB1;
    constexpr int NE = 4 * NJ;                      // accumulator elements per thread (per h: 2*NJ*2)
    const int n_promo_threads = 128 * C::ACTIVE_WGS;
    const int ptid = threadIdx.x - 256;
    if (wg < C::ACTIVE_WGS) {
      int ss = 0, accb = 0;
      uint32_t sph = 0, accph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = load_item(P, it, debug);
        const int n_tile = w.tile / P.n_m_tiles, m_tile = w.tile % P.n_m_tiles;
        const int m0 = m_tile * NT, n0 = n_tile * kTileW;
        const bool owner = (w.flags & 2) != 0;
        const bool split = (w.flags & 1) != 0;
        // acc index: ((h*2 + i)*NJ + j)*2 + e
        float acc[2 * NE];
        int32_t dacc[DEBUG ? 2 * NE : 1];
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const int64_t m = m0 + col0 + 8 * j + 2 * t0 + e;
            const float c0 = (owner && m < P.Mp) ? -__ldg(P.corr + m) * 0.001953125f : 0.f;   // 2^-9
#pragma unroll
            for (int hi = 0; hi < 4; ++hi) {
              acc[(hi * NJ + j) * 2 + e] = c0;
              if (DEBUG) dacc[(hi * NJ + j) * 2 + e] = 0;
            }
          }
        }
        for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
          const bool is8 = lds_u8(s_tags_a + kb) != 0;
          mbar_wait(&s_full[ss], sph);
          float2 sc[NJ];
          {
            const uint32_t sbase = sS_a + (ss * NT + col0 + 2 * t0) * 4;
#pragma unroll
            for (int j = 0; j < NJ; ++j) {
              const uint2 u = lds64(sbase + j * 32);
              sc[j] = make_float2(__uint_as_float(u.x), __uint_as_float(u.y));
            }
          }
          mbar_wait(&acc_full[accb], accph);
          tc_fence_after();
          const uint32_t tcol = tbase + kAccCol + accb * NT + col0;
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const uint32_t taddr = tcol + ((uint32_t)(32 * q + 16 * h) << 16);
#pragma unroll
            for (int part = 0; part < 2; ++part) {
              constexpr int dummy = 0;
              (void)dummy;
              const int jb = part == 0 ? 0 : NB1;
              const int nrep = part == 0 ? NB1 : NB2;
              if (nrep == 0) continue;
              uint32_t v[4 * 8];
              if (part == 0) tmem_ld_16x256b<NB1>(taddr, v);
              else if constexpr (NB2 > 0) tmem_ld_16x256b<(NB2 > 0 ? NB2 : 2)>(taddr + NB1 * 8, v);
              tmem_wait_ld();
              if (!is8) {
#pragma unroll
                for (int jj = 0; jj < 8; ++jj) {
                  if (jj < nrep) {
                    const int j = jb + jj;
#pragma unroll
                    for (int i = 0; i < 2; ++i) {
                      const int a = ((h * 2 + i) * NJ + j) * 2;
                      float2 y = ffma2(make_float2(__uint_as_float(v[4 * jj + 2 * i]), __uint_as_float(v[4 * jj + 2 * i + 1])),
                                       sc[j], make_float2(acc[a], acc[a + 1]));
                      acc[a] = y.x;
                      acc[a + 1] = y.y;
                    }
                  }
                }
              } else {
#pragma unroll
                for (int jj = 0; jj < 8; ++jj) {
                  if (jj < nrep) {
                    const int j = jb + jj;
                    const float2 s8 = make_float2(sc[j].x * 1.220703125e-04f, sc[j].y * 1.220703125e-04f);  // 2^-13
#pragma unroll
                    for (int i = 0; i < 2; ++i) {
                      const int a = ((h * 2 + i) * NJ + j) * 2;
                      float2 y = ffma2(make_float2(__int2float_rn((int)v[4 * jj + 2 * i]), __int2float_rn((int)v[4 * jj + 2 * i + 1])),
                                       s8, make_float2(acc[a], acc[a + 1]));
                      acc[a] = y.x;
                      acc[a + 1] = y.y;
                    }
                  }
                }
              }
              if (DEBUG) {
#pragma unroll
                for (int jj = 0; jj < 8; ++jj) {
                  if (jj < nrep) {
                    const int j = jb + jj;
#pragma unroll
                    for (int i = 0; i < 2; ++i) {
#pragma unroll
                      for (int e = 0; e < 2; ++e) {
                        const int64_t m = m0 + col0 + 8 * j + 2 * t0 + e;
                        const int n = n0 + 32 * q + 16 * h + t1 + 8 * i;
                        const uint32_t raw = v[4 * jj + 2 * i + e];
                        int32_t ab;
                        if (is8) {
                          ab = ((int32_t)raw) >> 4;
                        } else {
                          const int qs = (m < P.Mp) ? (int)P.qsum[(int64_t)kb * P.Mp + m] : 0;
                          ab = (int32_t)(__uint_as_float(raw) * 512.f) - 8 * qs;
                        }
                        dacc[((h * 2 + i) * NJ + j) * 2 + e] += ab;
                        if (DEBUG == 2 && m < P.M) P.dbg_blocks[((int64_t)kb * P.M + m) * P.N + n] = ab;
                      }
                    }
                  }
                }
              }
            }
          }
          tc_fence_before();
          __syncwarp();
          if (lane == 0) {
            mbar_arrive(&acc_empty[accb]);
            mbar_arrive(&s_empty[ss]);
          }
          if (++ss == kSRing) { ss = 0; sph ^= 1; }
          if (++accb == NACC) { accb = 0; accph ^= 1; }
        }
        // ---------------------------------------------------------------- epilogue
        if (split) {
          const int seg = (w.flags >> 8) & 0xFF;
          const int nseg = (w.flags >> 16) & 0xFF;
          const int64_t part_tile = (int64_t)NT * kTileW;    // = n_promo_threads * 2*NE floats
          if (!owner) {
            float4* dst = reinterpret_cast<float4*>(
                P.ws_part + ((int64_t)w.fix * (P.max_seg - 1) + (seg - 1)) * part_tile + (int64_t)ptid * 2 * NE);
#pragma unroll
            for (int a = 0; a < 2 * NE; a += 4) dst[a / 4] = make_float4(acc[a], acc[a + 1], acc[a + 2], acc[a + 3]);
            __threadfence();
            named_bar_sync(1, n_promo_threads);
            if (threadIdx.x == 256) st_release_gpu(P.ws_flags + (int64_t)w.fix * P.max_seg + seg, P.epoch);
            continue;
          }
          if (threadIdx.x == 256) {
            for (int sgi = 1; sgi < nseg; ++sgi) {
              const uint32_t* f = P.ws_flags + (int64_t)w.fix * P.max_seg + sgi;
              uint64_t t0g = globaltimer_ns();
              while (ld_acquire_gpu(f) != P.epoch) {
                if (globaltimer_ns() - t0g > COMET_MBAR_TIMEOUT_NS) {
                  __trap();
                }
              }
            }
          }
          named_bar_sync(1, n_promo_threads);
          for (int sgi = 1; sgi < nseg; ++sgi) {
            const float4* src = reinterpret_cast<const float4*>(
                P.ws_part + ((int64_t)w.fix * (P.max_seg - 1) + (sgi - 1)) * part_tile + (int64_t)ptid * 2 * NE);
#pragma unroll
            for (int a = 0; a < 2 * NE; a += 4) {
              float4 t4;
              asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];"
                           : "=f"(t4.x), "=f"(t4.y), "=f"(t4.z), "=f"(t4.w) : "l"(src + a / 4));
              acc[a] += t4.x; acc[a + 1] += t4.y; acc[a + 2] += t4.z; acc[a + 3] += t4.w;
            }
          }
        }
#pragma unroll
        for (int hi = 0; hi < 4; ++hi) {
          const int h = hi >> 1, i = hi & 1;
          const int n = n0 + 32 * q + 16 * h + t1 + 8 * i;
          const float swv = __ldg(P.w_scales + n) * 512.f;
#pragma unroll
          for (int j = 0; j < NJ; ++j) {
#pragma unroll
            for (int e = 0; e < 2; ++e) {
              const int64_t m = m0 + col0 + 8 * j + 2 * t0 + e;
              if (m < P.M) {
                const int a = (hi * NJ + j) * 2 + e;
                const float yv = acc[a] * swv;
                const int64_t off = m * P.ldy + n;
                if (P.ydt == COMET_F16) reinterpret_cast<__half*>(P.y)[off] = __float2half_rn(yv);
                else if (P.ydt == COMET_BF16) reinterpret_cast<__nv_bfloat16*>(P.y)[off] = __float2bfloat16_rn(yv);
                else reinterpret_cast<float*>(P.y)[off] = yv;
                if (DEBUG) P.dbg_acc[m * P.N + n] = dacc[a];
              }
            }
          }
        }
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (warp == 2) tmem_dealloc<512>(tbase);
}

template <int NT, int DEBUG>
cudaError_t launch_nt(const GemmParams& prm, int grid, cudaStream_t stream) {
  using C = Cfg<NT>;
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(k_w4ax<NT, DEBUG>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM_BYTES);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  k_w4ax<NT, DEBUG><<<grid, kThreads, C::SMEM_BYTES, stream>>>(prm);
  return cudaGetLastError();
}

PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

}  // namespace

// ------------------------------------------------------------------------------ host side
bool make_map_2d(CUtensorMap* map, const void* base, uint64_t inner, uint64_t outer,
                 uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer,
                 CUtensorMapSwizzle swz) {
  auto fn = encode_fn();
  if (!fn) return false;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {row_bytes};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, const_cast<void*>(base), dims, strides, box,
                  estr, CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

unsigned long long* g_trace = nullptr;

}  // namespace gemm

comet_status_t launch_gemm(Plan& p, const void* act_packed, const float* act_scales,
                           const void* w_packed, const float* w_scales, void* y,
                           comet_dtype_t ydt, int64_t ldy, int32_t* debug_acc,
                           int32_t* debug_acc_blocks, void* workspace, size_t ws_bytes,
                           cudaStream_t stream, int* launches) {
  using namespace gemm;
  *launches = 0;
  const bool dbg = debug_acc != nullptr || debug_acc_blocks != nullptr;
  const int debug = debug_acc_blocks ? 2 : (dbg ? 1 : 0);
  const bool normal = p.orientation >= 2;
  const int cg = p.orientation == 3 ? 2 : 1;
  // token-tile and weight-tile of one CTA (= box rows of the two TMA maps) and of the tile
  int tile_m, tile_w, cta_rows_w;
  if (normal) { tile_m = 128 * cg; tile_w = dbg ? 96 : p.tile_w; cta_rows_w = tile_w / cg; }
  else { tile_m = dbg ? 64 : p.tile_n; tile_w = kTileW; cta_rows_w = kTileW; }
  const int box_m = normal ? 128 : tile_m;
  comet_act_layout_t L;
  act_layout(p.M, p.K, &L);
  const uint8_t* base = static_cast<const uint8_t*>(act_packed);
  GemmParams prm;
  memset(&prm, 0, sizeof(prm));
  if (!make_map_2d(&prm.map_x, base + L.codes_off, (uint64_t)p.K, (uint64_t)p.M, (uint64_t)p.K, 128,
                   (uint32_t)box_m, CU_TENSOR_MAP_SWIZZLE_128B))
    return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the activation codes");
  if (!make_map_2d(&prm.map_w, w_packed, (uint64_t)(p.K / 2), (uint64_t)p.N, (uint64_t)(p.K / 2), 64,
                   (uint32_t)cta_rows_w, CU_TENSOR_MAP_SWIZZLE_64B))
    return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the packed weights");
  if (normal && !dbg) {
    const int esz = ydt == COMET_F32 ? 4 : 2;
    if (!make_map_2d(&prm.map_y, y, (uint64_t)p.N * esz, (uint64_t)p.M, (uint64_t)ldy * esz, 64, 128,
                     CU_TENSOR_MAP_SWIZZLE_64B))
      return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the output");
  }
  prm.scales = act_scales;
  prm.corr = reinterpret_cast<const float*>(base + L.corr_off);
  prm.qsum = reinterpret_cast<const int16_t*>(base + L.qsum_off);
  prm.w_scales = w_scales;
  prm.y = y;
  prm.ldy = ldy;
  prm.dbg_acc = debug_acc;
  prm.dbg_blocks = debug_acc_blocks;
  prm.M = p.M;
  prm.N = p.N;
  prm.Mp = L.Mp;
  prm.nb = (int)p.nb;
  prm.ydt = (int)ydt;
  prm.tags = p.mask;
  {
    const char* ab = getenv("COMET_ABLATE");
    prm.ablate = ab ? atoi(ab) : 0;
    prm.trace = g_trace;
  }
  cudaError_t e;
  int grid;
  if (dbg) {
    // whole tiles, one CTA each, narrower tiles (the debug accumulators need the registers)
    prm.n_m_tiles = (int)ceil_div(p.M, tile_m);
    grid = (int)(prm.n_m_tiles * ceil_div(p.N, tile_w)) * cg;
    prm.max_seg = 1;
  } else {
    if (p.d_items == nullptr) return fail(COMET_ERR_INVALID_ARG, "plan was created with device_plan = 0");
    if (p.ws_bytes > 0 && (workspace == nullptr || ws_bytes < p.ws_bytes))
      return fail(COMET_ERR_WORKSPACE_TOO_SMALL, "workspace smaller than the plan's workspace_bytes");
    prm.n_m_tiles = (int)p.n_m_tiles;
    prm.cta_begin = p.d_cta_begin;
    prm.items = p.d_items;
    prm.max_seg = p.max_segments;
    prm.ws_part = static_cast<float*>(workspace);
    prm.ws_flags = reinterpret_cast<uint32_t*>(static_cast<uint8_t*>(workspace) + p.ws_flags_off);
    prm.epoch = ++p.epoch;
    grid = p.num_ctas * cg;
  }
  if (normal) {
    e = launch_gemm_n(prm, grid, tile_w, cg, debug, stream);
  } else if (dbg) {
    e = debug == 2 ? launch_nt<64, 2>(prm, grid, stream) : launch_nt<64, 1>(prm, grid, stream);
  } else {
    switch (tile_m) {
      case 16: e = launch_nt<16, 0>(prm, grid, stream); break;
      case 32: e = launch_nt<32, 0>(prm, grid, stream); break;
      case 64: e = launch_nt<64, 0>(prm, grid, stream); break;
      case 128: e = launch_nt<128, 0>(prm, grid, stream); break;
      case 192: e = launch_nt<192, 0>(prm, grid, stream); break;
      case 224: e = launch_nt<224, 0>(prm, grid, stream); break;
      default: return fail(COMET_ERR_UNSUPPORTED_SHAPE, "unsupported tile_n");
    }
  }
  if (e != cudaSuccess) return cuda_status(e, "w4ax gemm launch");
  *launches = 1;
  return COMET_OK;
}

}  // namespace comet
