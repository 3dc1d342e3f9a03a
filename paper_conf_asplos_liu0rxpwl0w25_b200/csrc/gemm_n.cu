// gemm_n.cu -- the W4Ax GEMM with TOKENS on the MMA M side (prefill-sized M).
//
//   Y[m, n] = s_w[n] * sum_b s_a[m,b] * acc_b[m,n]
//
// Output tile: 128 tokens (MMA M = TMEM lanes) x BN weights (MMA N = TMEM columns, BN = 256).
// A operand = the activation tile, TMA-staged straight from the mixed-precision code plane
// (E4M3 bytes for INT4 blocks, s8 for INT8 blocks; 128-byte swizzle, no conversion).
// B operand = the weight tile, widened from packed INT4 by CUDA cores into a 128-byte-swizzled
// K-major shared-memory buffer (the paper's "convert on CUDA cores, store the converted result
// directly in shared memory"), double-buffered so widening of K-block b+1 overlaps the
// MMA of K-block b (the SIMT-enhanced pipeline).
// Promotion ("dequant"): TMEM lane = token, so every promotion thread needs exactly ONE
// activation scale s_a[m,b] per K-block and folds the 32x32b-loaded FP32 accumulator row into
// its registers with FFMA2 (two columns per instruction).
//
// Roles (512 threads): warp 0 TMA producer, warp 1 MMA issuer, warp 2 TMEM allocator,
// warps 4-7 widen, warps 8-15 promotion + epilogue (two warpgroups, BN/2 columns each).
//
// CG = 2 (CTA pair, tcgen05 cta_group::2): the tile is 256 tokens x BN weights; CTA r of the
// pair holds tokens m0 + 128 r (its half of A, its TMEM lanes) and widens weights
// n0 + r BN/2 .. (its half of B), so each SM widens half as many weight rows per MMA FLOP.
// The even CTA issues the pair MMA; both CTAs' widen / promotion warps arrive on the even
// CTA's b_full / acc_empty barriers, MMA completion is multicast to both CTAs.
#include "gemm_common.cuh"

namespace comet {
namespace gemm {
namespace {

template <int BN, int CG>
struct CfgN {
  static constexpr int BM = 128;                          // tokens per CTA (TMEM lanes)
  static constexpr int WROWS = BN / CG;                   // weight rows widened by this CTA
  static constexpr int X_BYTES = BM * 128;                // activation tile (one K-block)
  static constexpr int WP_BYTES = WROWS * 64;             // packed weight rows
  static constexpr int STAGE_BYTES = X_BYTES + WP_BYTES;
  static constexpr int B_BYTES = WROWS * 128;             // widened weight rows (MMA B half)
  static constexpr int NBUF = 2;                          // widened-weight ring
  static constexpr int COLS = BN / 2;                     // accumulator columns per promotion WG
  static constexpr int NACC = (3 * BN <= 512) ? 3 : 2;    // accumulators in TMEM
  static constexpr int ROWS_PER_THREAD = (WROWS + 127) / 128;   // widen rows per thread
  static constexpr int STAGES_RAW = (200 * 1024 - NBUF * B_BYTES - kSRing * BM * 4) / STAGE_BYTES;
  static constexpr int STAGES = STAGES_RAW > 8 ? 8 : STAGES_RAW;
  static constexpr int SMEM_DATA = STAGES * STAGE_BYTES + NBUF * B_BYTES + kSRing * BM * 4;
  static constexpr int N_BARS = 2 * STAGES + 2 * NBUF + 2 * NACC + 2 * kSRing;
  static constexpr int SMEM_BYTES = 1024 + SMEM_DATA + N_BARS * 8 + 16 + kMaxBlocks;
  static_assert(STAGES >= 2, "pipeline depth");
  static_assert(NACC * BN <= 512, "TMEM budget");
  static_assert(COLS % 32 == 0, "promotion batches");
};

template <int BN, int CG, int DEBUG>
__global__ void __launch_bounds__(kThreads, 1) k_w4ax_n(const __grid_constant__ GemmParams P) {
  using C = CfgN<BN, CG>;
  constexpr int S = C::STAGES;
  constexpr int NACC = C::NACC;
  constexpr int BM = C::BM;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint8_t* sX = smem;                                     // [S][BM x 128 B]   (A)
  uint8_t* sWp = sX + S * C::X_BYTES;                     // [S][BN x 64 B]    packed W
  uint8_t* sB = sWp + S * C::WP_BYTES;                    // [NBUF][BN x 128 B] widened W (B)
  float* sS = reinterpret_cast<float*>(sB + C::NBUF * C::B_BYTES);   // [kSRing][BM]
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::SMEM_DATA);
  uint64_t* full = bars;                     // [S]     TMA -> MMA, widen
  uint64_t* empty = full + S;                // [S]     MMA commit + 4 widen warps -> TMA
  uint64_t* b_full = empty + S;              // [NBUF]  widen -> MMA
  uint64_t* b_empty = b_full + C::NBUF;      // [NBUF]  MMA commit -> widen
  uint64_t* acc_full = b_empty + C::NBUF;    // [NACC]  MMA commit -> promotion
  uint64_t* acc_empty = acc_full + NACC;     // [NACC]  promotion -> MMA
  uint64_t* s_full = acc_empty + NACC;       // [kSRing]
  uint64_t* s_empty = s_full + kSRing;       // [kSRing]
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + C::N_BARS);
  uint8_t* s_tags = reinterpret_cast<uint8_t*>(tmem_holder + 4);
  const uint32_t s_tags_a = smem_u32(s_tags);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const bool debug = DEBUG != 0;
  const uint32_t rank = CG == 2 ? cluster_ctarank() : 0;   // CTA rank within the pair
  const int unit = blockIdx.x / CG;                          // work list index (pair or CTA)
  const int it_begin = debug ? unit : P.cta_begin[unit];
  const int it_end = debug ? unit + 1 : P.cta_begin[unit + 1];
  const int nb = P.nb;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&P.map_x);
    tma_prefetch(&P.map_w);
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1 + 4);
    }
    for (int i = 0; i < C::NBUF; ++i) {
      mbar_init(&b_full[i], 4 * CG);
      mbar_init(&b_empty[i], 1);
    }
    for (int i = 0; i < NACC; ++i) {
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_empty[i], 8 * CG);
    }
    for (int i = 0; i < kSRing; ++i) {
      mbar_init(&s_full[i], 1);
      mbar_init(&s_empty[i], 8);
    }
    fence_mbar_init();
  }
  if (warp == 2) {
    if (CG == 2) { tmem_alloc_cg2<512>(tmem_holder); tmem_relinquish_cg2(); }
    else { tmem_alloc<512>(tmem_holder); tmem_relinquish(); }
  }
  for (int i = threadIdx.x; i < nb; i += kThreads) s_tags[i] = P.tags.get(i) ? 1 : 0;
  tc_fence_before();
  __syncthreads();
  if (CG == 2) cluster_sync();                 // peer barriers initialised before remote arrives
  tc_fence_after();
  const uint32_t tbase = *tmem_holder;
  // the even CTA's barriers that both CTAs arrive on (shared::cluster addresses)
  const uint32_t b_full_lead = CG == 2 ? mapa_shared(smem_u32(b_full), 0) : smem_u32(b_full);
  const uint32_t acc_empty_lead = CG == 2 ? mapa_shared(smem_u32(acc_empty), 0) : smem_u32(acc_empty);
  auto wait_x = [&](uint64_t* bar, uint32_t par) { mbar_wait(bar, par); };

  if (warp < 4) {
    setmaxnreg_dec<32>();
    if (warp == 0 && lane == 0) {
      // ------------------------------------------------------------------ TMA producer
      int stage = 0, ss = 0;
      uint32_t ph = 0, sph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = load_item(P, it, debug);
        const int n_tile = w.tile / P.n_m_tiles, m_tile = w.tile % P.n_m_tiles;
        const int m0 = m_tile * (BM * CG) + BM * rank, n0 = n_tile * BN + C::WROWS * rank;
        const uint32_t sbytes = m0 < P.Mp ? (uint32_t)(min((int64_t)BM, P.Mp - m0) * 4) : 0u;
        for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
          wait_x(&empty[stage], ph ^ 1);
          mbar_arrive_expect_tx(&full[stage], C::STAGE_BYTES);
          tma_load_2d(sX + stage * C::X_BYTES, &P.map_x, &full[stage], kb * 128, m0);
          tma_load_2d(sWp + stage * C::WP_BYTES, &P.map_w, &full[stage], kb * 64, n0);
          mbar_wait(&s_empty[ss], sph ^ 1);
          if (sbytes) {
            mbar_arrive_expect_tx(&s_full[ss], sbytes);
            bulk_load(sS + ss * BM, P.scales + (int64_t)kb * P.Mp + m0, sbytes, &s_full[ss]);
          } else {
            mbar_arrive(&s_full[ss]);        // this CTA's tokens are all padding
          }
          if (++stage == S) { stage = 0; ph ^= 1; }
          if (++ss == kSRing) { ss = 0; sph ^= 1; }
        }
      }
    } else if (warp == 1 && lane == 0 && rank == 0) {
      // ------------------------------------------------------------------ MMA issuer
      const uint32_t id_f8 = idesc_f8f6f4_e4m3(BM * CG, BN);
      const uint32_t id_i8 = idesc_i8(BM * CG, BN);
      int stage = 0, bb = 0, accb = 0;
      uint32_t ph = 0, bph = 0, accph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = load_item(P, it, debug);
        for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
          wait_x(&acc_empty[accb], accph ^ 1);
          // b_full covers the stage too: every widen warp waited on its CTA's full[stage]
          wait_x(&b_full[bb], bph);
          tc_fence_after();
          const uint32_t d = tbase + accb * BN;
          const uint32_t sa = smem_u32(sX + stage * C::X_BYTES);
          const uint32_t sbv = smem_u32(sB + bb * C::B_BYTES);
          if (lds_u8(s_tags_a + kb)) {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const uint64_t ad = sdesc_kmajor_sw128(sa + 32 * k), bd = sdesc_kmajor_sw128(sbv + 32 * k);
              if (CG == 2) mma_i8_ss_cg2(d, ad, bd, id_i8, k); else mma_i8_ss(d, ad, bd, id_i8, k);
            }
          } else {
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const uint64_t ad = sdesc_kmajor_sw128(sa + 32 * k), bd = sdesc_kmajor_sw128(sbv + 32 * k);
              if (CG == 2) mma_f8_ss_cg2(d, ad, bd, id_f8, k); else mma_f8_ss(d, ad, bd, id_f8, k);
            }
          }
          if (CG == 2) {
            tc_commit_mc(&empty[stage], 3);
            tc_commit_mc(&b_empty[bb], 3);
            tc_commit_mc(&acc_full[accb], 3);
          } else {
            tc_commit(&empty[stage]);
            tc_commit(&b_empty[bb]);
            tc_commit(&acc_full[accb]);
          }
          if (++stage == S) { stage = 0; ph ^= 1; }
          if (++bb == C::NBUF) { bb = 0; bph ^= 1; }
          if (++accb == NACC) { accb = 0; accph ^= 1; }
        }
      }
    }
  } else if (warp < 8) {
    setmaxnreg_dec<64>();
    // -------------------------------------------------------------------- widen (W -> smem B)
    const int t = threadIdx.x - 128;                      // weight row t (and t + 128)
    const bool has_row = t < C::WROWS;
    const uint32_t sWp_a = smem_u32(sWp), sB_a = smem_u32(sB);
    int stage = 0, bb = 0;
    uint32_t ph = 0, bph = 0;
    for (int it = it_begin; it < it_end; ++it) {
      const WorkItem w = load_item(P, it, debug);
      for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
        const bool is8 = lds_u8(s_tags_a + kb) != 0;
        wait_x(&full[stage], ph);
        uint4 c[C::ROWS_PER_THREAD][4];
#pragma unroll
        for (int rr = 0; rr < C::ROWS_PER_THREAD; ++rr) {
          const int row = t + 128 * rr;
          const uint32_t src = sWp_a + stage * C::WP_BYTES + row * 64;
          const int sw = (row >> 1) & 3;                  // TMA 64-byte swizzle
#pragma unroll
          for (int j = 0; j < 4; ++j) c[rr][j] = has_row ? lds128(src + ((j ^ sw) << 4)) : make_uint4(0, 0, 0, 0);
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[stage]);
        wait_x(&b_empty[bb], bph ^ 1);
#pragma unroll
        for (int rr = 0; rr < C::ROWS_PER_THREAD; ++rr) {
          if (!has_row) break;
          const int row = t + 128 * rr;
          const uint32_t dst = sB_a + bb * C::B_BYTES + row * 128;
          const int sw = row & 7;                         // UMMA/TMA 128-byte swizzle
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const uint32_t pw[4] = {c[rr][j].x, c[rr][j].y, c[rr][j].z, c[rr][j].w};
            uint32_t o[8];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const uint32_t p = pw[i];
              if (is8) {
                o[2 * i] = ((p << 4) & 0xF0F0F0F0u) ^ 0x80808080u;
                o[2 * i + 1] = (p & 0xF0F0F0F0u) ^ 0x80808080u;
              } else {
                o[2 * i] = p & 0x0F0F0F0Fu;
                o[2 * i + 1] = (p >> 4) & 0x0F0F0F0Fu;
              }
            }
            // logical 16-byte chunks 2j and 2j+1 (channels 32j .. 32j+31)
            asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(dst + (((2 * j) ^ sw) << 4)),
                         "r"(o[0]), "r"(o[1]), "r"(o[2]), "r"(o[3]) : "memory");
            asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(dst + (((2 * j + 1) ^ sw) << 4)),
                         "r"(o[4]), "r"(o[5]), "r"(o[6]), "r"(o[7]) : "memory");
          }
        }
        fence_proxy_async_smem();                         // generic-proxy stores -> tensor core
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(b_full_lead + bb * 8);
        if (++stage == S) { stage = 0; ph ^= 1; }
        if (++bb == C::NBUF) { bb = 0; bph ^= 1; }
      }
    }
  } else {
    setmaxnreg_inc<208>();
    // -------------------------------------------------------------------- promotion + epilogue
    const int wg = (warp - 8) >> 2;
    const int q = warp & 3;
    const int r = q * 32 + lane;                          // TMEM lane = token row within the tile
    const uint32_t lane_addr = (uint32_t)(q * 32) << 16;
    constexpr int COLS = C::COLS;
    constexpr int BC = COLS > 64 ? 64 : COLS;             // columns per TMEM load batch
    constexpr int NBATCH = COLS / BC;
    const int col0 = wg * COLS;
    const int ptid = threadIdx.x - 256;
    const uint32_t sS_a = smem_u32(sS);
    int ss = 0, accb = 0;
    uint32_t sph = 0, accph = 0;
    for (int it = it_begin; it < it_end; ++it) {
      const WorkItem w = load_item(P, it, debug);
      const int n_tile = w.tile / P.n_m_tiles, m_tile = w.tile % P.n_m_tiles;
      const int m0 = m_tile * (BM * CG) + BM * rank, n0 = n_tile * BN;
      const int64_t m = m0 + r;
      const bool owner = (w.flags & 2) != 0;
      const bool split = (w.flags & 1) != 0;
      const float init = (owner && m < P.Mp) ? -__ldg(P.corr + m) * 0.001953125f : 0.f;   // 2^-9
      float acc[COLS];
      int32_t dacc[DEBUG ? COLS : 1];
#pragma unroll
      for (int c = 0; c < COLS; ++c) {
        acc[c] = init;
        if (DEBUG) dacc[c] = 0;
      }
      for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
        const bool is8 = lds_u8(s_tags_a + kb) != 0;
        mbar_wait(&s_full[ss], sph);
        float s;
        asm volatile("ld.shared.f32 %0, [%1];" : "=f"(s) : "r"(sS_a + (ss * BM + r) * 4));
        if (is8) s *= 1.220703125e-04f;                   // 2^-13: INT8 block acc = 16 sum x w
        const float2 s2 = make_float2(s, s);
        int qs = 0;
        if (DEBUG && !is8 && m < P.Mp) qs = P.qsum[(int64_t)kb * P.Mp + m];
        wait_x(&acc_full[accb], accph);
        tc_fence_after();
        const uint32_t taddr = tbase + accb * BN + col0 + lane_addr;
#pragma unroll
        for (int b = 0; b < NBATCH; ++b) {
          uint32_t v[BC];
          tmem_ld_32x32b<BC>(taddr + b * BC, v);
          tmem_wait_ld();
          if (DEBUG) {
#pragma unroll
            for (int c = 0; c < BC; ++c) {
              const int32_t ab = is8 ? (((int32_t)v[c]) >> 4) : ((int32_t)(__uint_as_float(v[c]) * 512.f) - 8 * qs);
              dacc[b * BC + c] += ab;
              if (DEBUG == 2 && m < P.M && n0 + col0 + b * BC + c < P.N)
                P.dbg_blocks[((int64_t)kb * P.M + m) * P.N + n0 + col0 + b * BC + c] = ab;
            }
          }
          if (is8) {
#pragma unroll
            for (int c = 0; c < BC; ++c) v[c] = __float_as_uint(__int2float_rn((int)v[c]));
          }
#pragma unroll
          for (int c = 0; c < BC; c += 2) {
            const int a = b * BC + c;
            float2 y = ffma2(make_float2(__uint_as_float(v[c]), __uint_as_float(v[c + 1])), s2,
                             make_float2(acc[a], acc[a + 1]));
            acc[a] = y.x;
            acc[a + 1] = y.y;
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          mbar_arrive_cluster(acc_empty_lead + accb * 8);
          mbar_arrive(&s_empty[ss]);
        }
        if (++ss == kSRing) { ss = 0; sph ^= 1; }
        if (++accb == NACC) { accb = 0; accph ^= 1; }
      }
      // ---------------------------------------------------------------- epilogue
      if (split) {
        const int seg = (w.flags >> 8) & 0xFF;
        const int nseg = (w.flags >> 16) & 0xFF;
        const int64_t part_tile = (int64_t)BM * BN;        // = 256 threads * COLS floats
        if (!owner) {
          float4* dst = reinterpret_cast<float4*>(
              P.ws_part + (((int64_t)w.fix * (P.max_seg - 1) + (seg - 1)) * CG + rank) * part_tile + (int64_t)ptid * COLS);
#pragma unroll
          for (int a = 0; a < COLS; a += 4) dst[a / 4] = make_float4(acc[a], acc[a + 1], acc[a + 2], acc[a + 3]);
          __threadfence();
          named_bar_sync(1, 256);
          if (threadIdx.x == 256) st_release_gpu(P.ws_flags + ((int64_t)w.fix * P.max_seg + seg) * CG + rank, P.epoch);
          continue;
        }
        if (threadIdx.x == 256) {
          for (int sgi = 1; sgi < nseg; ++sgi) {
            const uint32_t* f = P.ws_flags + ((int64_t)w.fix * P.max_seg + sgi) * CG + rank;
            uint64_t t0g = globaltimer_ns();
            while (ld_acquire_gpu(f) != P.epoch) {
              if (globaltimer_ns() - t0g > COMET_MBAR_TIMEOUT_NS) {
                printf("comet: stream-K fix-up timeout (tile %d seg %d)\n", w.tile, sgi);
                __trap();
              }
            }
          }
        }
        named_bar_sync(1, 256);
        for (int sgi = 1; sgi < nseg; ++sgi) {
          const float4* src = reinterpret_cast<const float4*>(
              P.ws_part + (((int64_t)w.fix * (P.max_seg - 1) + (sgi - 1)) * CG + rank) * part_tile + (int64_t)ptid * COLS);
#pragma unroll
          for (int a = 0; a < COLS; a += 4) {
            float4 t4;
            asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];"
                         : "=f"(t4.x), "=f"(t4.y), "=f"(t4.z), "=f"(t4.w) : "l"(src + a / 4));
            acc[a] += t4.x; acc[a + 1] += t4.y; acc[a + 2] += t4.z; acc[a + 3] += t4.w;
          }
        }
      }
      const int nbase = n0 + col0;
      if (m < P.M && nbase < P.N) {
        const float* swp = P.w_scales + nbase;
        if (P.ydt == COMET_F32) {
          float* yrow = reinterpret_cast<float*>(P.y) + m * P.ldy + nbase;
#pragma unroll
          for (int c = 0; c < COLS; c += 4) {
            const float4 sw4 = __ldg(reinterpret_cast<const float4*>(swp + c));
            reinterpret_cast<float4*>(yrow)[c / 4] = make_float4(acc[c] * sw4.x * 512.f, acc[c + 1] * sw4.y * 512.f,
                                                                 acc[c + 2] * sw4.z * 512.f, acc[c + 3] * sw4.w * 512.f);
          }
        } else {
          uint16_t* yrow = reinterpret_cast<uint16_t*>(P.y) + m * P.ldy + nbase;
          const bool bf = P.ydt == COMET_BF16;
#pragma unroll
          for (int c = 0; c < COLS; c += 8) {
            const float4 sa = __ldg(reinterpret_cast<const float4*>(swp + c));
            const float4 sb = __ldg(reinterpret_cast<const float4*>(swp + c + 4));
            const float f[8] = {acc[c] * sa.x * 512.f, acc[c + 1] * sa.y * 512.f, acc[c + 2] * sa.z * 512.f,
                                acc[c + 3] * sa.w * 512.f, acc[c + 4] * sb.x * 512.f, acc[c + 5] * sb.y * 512.f,
                                acc[c + 6] * sb.z * 512.f, acc[c + 7] * sb.w * 512.f};
            uint32_t pk[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              if (bf) {
                __nv_bfloat162 h = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
                pk[i] = *reinterpret_cast<uint32_t*>(&h);
              } else {
                __half2 h = __floats2half2_rn(f[2 * i], f[2 * i + 1]);
                pk[i] = *reinterpret_cast<uint32_t*>(&h);
              }
            }
            reinterpret_cast<uint4*>(yrow)[c / 8] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
          }
        }
        if (DEBUG) {
#pragma unroll
          for (int c = 0; c < COLS; ++c) P.dbg_acc[m * P.N + nbase + c] = dacc[c];
        }
      }
    }
  }

  tc_fence_before();
  __syncthreads();
  if (CG == 2) cluster_sync();                 // the pair is done with each other's smem / TMEM
  if (warp == 2) {
    if (CG == 2) tmem_dealloc_cg2<512>(tbase); else tmem_dealloc<512>(tbase);
  }
}

template <int BN, int CG, int DEBUG>
cudaError_t launch_bn(const GemmParams& prm, int grid, cudaStream_t stream) {
  using C = CfgN<BN, CG>;
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(k_w4ax_n<BN, CG, DEBUG>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM_BYTES);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = C::SMEM_BYTES;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CG;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k_w4ax_n<BN, CG, DEBUG>, prm);
}

}  // namespace

cudaError_t launch_gemm_n(const GemmParams& prm, int grid, int bn, int cg, int debug, cudaStream_t stream) {
  if (cg == 2) {
    if (debug == 2) return launch_bn<128, 2, 2>(prm, grid, stream);
    if (debug == 1) return launch_bn<128, 2, 1>(prm, grid, stream);
    return launch_bn<256, 2, 0>(prm, grid, stream);
  }
  if (debug == 2) return launch_bn<128, 1, 2>(prm, grid, stream);
  if (debug == 1) return launch_bn<128, 1, 1>(prm, grid, stream);
  if (bn == 128) return launch_bn<128, 1, 0>(prm, grid, stream);
  return launch_bn<256, 1, 0>(prm, grid, stream);
}

}  // namespace gemm
}  // namespace comet
