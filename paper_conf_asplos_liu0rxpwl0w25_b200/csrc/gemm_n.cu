// gemm_n.cu -- the W4Ax GEMM with TOKENS on the MMA M side (prefill-sized M).
//
//   Y[m, n] = s_w[n] * sum_b s_a[m,b] * acc_b[m,n]
//
// Output tile: 128 tokens (MMA M = TMEM lanes) x BN weights (MMA N = TMEM columns, BN = 192
// or 256).
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
// Roles: warpgroup 0 = TMA producer (warp 0), two MMA issuers (warps 1, 3), TMEM allocator
// (warp 2); NWG widen warpgroups (taking K-blocks in turn); NPW promotion + epilogue
// warpgroups (BN / NPW accumulator columns each).
//
// CG = 2 (CTA pair, tcgen05 cta_group::2): the tile is 256 tokens x BN weights; CTA r of the
// pair holds tokens m0 + 128 r (its half of A, its TMEM lanes) and widens weights
// n0 + r BN/2 .. (its half of B), so each SM widens half as many weight rows per MMA FLOP.
// The even CTA issues the pair MMA; both CTAs' widen / promotion warps arrive on the even
// CTA's b_full / acc_empty barriers, MMA completion is multicast to both CTAs.
#include "gemm_common.cuh"

#ifndef COMET_ISSUERS
#define COMET_ISSUERS 2   // MMA issuing threads (K-blocks alternate between them)
#endif
#ifndef COMET_NSTAGE
#define COMET_NSTAGE 2   // output staging buffers per promotion warpgroup (TMA-store epilogue)
#endif
#ifndef COMET_N_UNIFORM_MMA
#define COMET_N_UNIFORM_MMA 1   // 1: MMA issue loop on the whole warp with uniform operands, one elected lane issues MMAs + commits
#endif
#ifndef COMET_PRODUCERS
#define COMET_PRODUCERS 1   // TMA-issuing warps (2: K-blocks alternate between them)
#endif
#ifndef COMET_PROMO_SB
#define COMET_PROMO_SB 1    // single-buffered 32-column promotion batches when they fit
#endif
#ifndef COMET_SPIN_MMA
#define COMET_SPIN_MMA 0    // 1: MMA issuers spin (test_wait) on mma_ready instead of suspending
#endif
#ifndef COMET_SPIN_PROMO
#define COMET_SPIN_PROMO 0  // 1: promotion warps spin on acc_full instead of suspending
#endif
#ifndef COMET_PROMO_W64
#define COMET_PROMO_W64 1   // 64-column TMEM load rounds in the promotion when the registers allow
#endif
#ifndef COMET_WIDEN40
#define COMET_WIDEN40 1     // widen warpgroups at 40 registers when promotion still fits
#endif
#ifndef COMET_NSUB
#define COMET_NSUB 1   // 2: split each K-block's MMA into two sub-MMAs (experimental, slower)
#endif
#ifndef COMET_SMEM_BUDGET_KB
#define COMET_SMEM_BUDGET_KB 216   // pipeline slots + output staging + scale ring
#endif
#ifndef COMET_PROMO_WAIT_PLAIN
#define COMET_PROMO_WAIT_PLAIN 1   // 1: promotion waits acc_full with a plain try_wait loop (see the wait)
#endif
#ifndef COMET_ABLATE_TMA2D
#define COMET_ABLATE_TMA2D 0   // 1: timing experiment only -- contiguous bulk copies from a small L2-resident buffer replace the 2D TMA loads (wrong results)
#endif
#ifndef COMET_MMA_WAIT_PLAIN
#define COMET_MMA_WAIT_PLAIN 1   // 1: MMA issuer waits mma_ready with a plain try_wait loop (iteration-count guard)
#endif
#ifndef COMET_WIDEN_WAIT_PLAIN
#define COMET_WIDEN_WAIT_PLAIN 0   // experiment: plain try_wait loop for the widen warps' full wait
#endif
#ifndef COMET_LDTM_X64
#define COMET_LDTM_X64 0   // 1: the promotion's 64-column rounds as one 32x32b.x64 load instead of two .x32
#endif
#ifndef COMET_PREWIDENED_UB
#define COMET_PREWIDENED_UB 0   // SURVEY §8(d) ablation, timing only: B arrives pre-widened by TMA (2x weight bytes), no widening work
#endif
#ifndef COMET_PROMO_SCALAR
#define COMET_PROMO_SCALAR 0    // SURVEY §8(d) ablation: scalar FFMA promotion instead of FFMA2
#endif
#ifndef COMET_STUB
#define COMET_STUB 0   // timing experiments only (wrong results): 1 MMA kind fixed, 2 promotion scale/kind fixed, 4 no scale loads, 8 no epilogue stores
#endif
#ifndef COMET_N256_SMEM_KB
#define COMET_N256_SMEM_KB COMET_SMEM_BUDGET_KB
#endif
#ifndef COMET_N256_NPW
#define COMET_N256_NPW 2   // promotion warpgroups of the 256-wide tile
#endif
#ifndef COMET_N256_NWG
#define COMET_N256_NWG 1   // widen warpgroups of the 256-wide tile (1: its registers go to promotion)
#endif

namespace comet {
namespace gemm {
namespace {

template <int BN, int CG, int NPW_, int NWG_, int DEBUG_, bool GS_ = false>
struct CfgN {
  static constexpr int BM = 128;                          // tokens per CTA (TMEM lanes)
  static constexpr int WROWS = BN / CG;                   // weight rows widened by this CTA
  static constexpr int X_BYTES = BM * 128;                // activation tile (one K-block)
  static constexpr int WP_BYTES = WROWS * 64;             // packed weight rows
  static constexpr int B_BYTES = WROWS * 128;             // widened weight rows (MMA B half)
  static constexpr int SLOT_BYTES = X_BYTES + WP_BYTES + B_BYTES;
  static constexpr int NPW = NPW_;                        // promotion warpgroups
  static constexpr int NWG = NWG_;                        // widen warpgroups (K-blocks in turn)
  static constexpr int THREADS = 128 * (1 + NWG + NPW);
  static constexpr int COLS = BN / NPW;                   // accumulator columns per promotion WG
  // setmaxnreg only redistributes the launch-time pool (THREADS x floor8(65536 / THREADS)):
  // the producer/MMA and widen warpgroups get REG_LOW (40, or 32 when that lets promotion fit
  // its working set), promotion the rest.
  static constexpr int REG_LAUNCH = ((65536 / THREADS) / 8) * 8;
  static constexpr int REG_POOL = REG_LAUNCH * (1 + NWG + NPW);
  static constexpr int promo_regs(int low) {
    return ((REG_POOL - low * (1 + NWG)) / NPW / 8) * 8 > 248 ? 248 : ((REG_POOL - low * (1 + NWG)) / NPW / 8) * 8;
  }
  static constexpr int ACC_REGS = COLS * (DEBUG_ ? 2 : 1);  // FP32 sums (+ debug int sums)
  // LOADALL: every column of the K-block is loaded with one wait, the accumulator released at
  // once, and the FFMA2 folding done afterwards; else 16/32-column batches double-buffered.
  static constexpr bool LOADALL = COLS <= 120 && promo_regs(32) >= ACC_REGS + COLS + 24;
  static constexpr int NEED_STD = LOADALL ? ACC_REGS + COLS + 24 : ACC_REGS + 2 * 16 + 24;
  // TIGHT: four promotion warpgroups (16 warps read TMEM: ~360 B/clk/SM against ~215 with 8,
  // profiles/r01/probe_b200.json) leave each promotion thread ~104 registers: the producer /
  // MMA warpgroup drops to 24, promotion folds single-buffered 16-column batches.
  static constexpr int promo_regs3(int low0, int loww) {
    return ((REG_POOL - low0 - loww * NWG) / NPW / 8) * 8 > 248 ? 248 : ((REG_POOL - low0 - loww * NWG) / NPW / 8) * 8;
  }
  static constexpr bool TIGHT = !LOADALL && promo_regs3(32, 32) < NEED_STD;
  static constexpr int NEED = TIGHT ? ACC_REGS + 16 + 24 : NEED_STD;
  static constexpr int REG_LOW = TIGHT ? 24 : (promo_regs(40) >= NEED ? 40 : 32);
  // the widen warpgroups keep 40 registers (their loop state spills at 32) whenever the
  // producer/MMA warpgroup at 32 still leaves promotion its working set
  static constexpr int promo_regs2(int low0, int loww) {
    return ((REG_POOL - low0 - loww * NWG) / NPW / 8) * 8 > 248 ? 248 : ((REG_POOL - low0 - loww * NWG) / NPW / 8) * 8;
  }
  static constexpr int REG_WIDEN = TIGHT ? 40 : ((REG_LOW == 32 && COMET_WIDEN40 && promo_regs2(32, 40) >= NEED) ? 40 : REG_LOW);
  static constexpr int REG_PROMO = promo_regs2(REG_LOW, REG_WIDEN);
  // SB: single-buffered 32-column batches (fewer, larger TMEM loads in flight) when the
  // double-buffered 32-column form does not fit (variant experiments: COMET_PROMO_SB)
  // W64: the accumulator leaves TMEM in 64-column rounds (two 32-column loads in flight, one
  // wait) -- half the load round trips of 32-column batches before the buffer is released
  static constexpr bool W64 = !LOADALL && !TIGHT && COLS % 64 == 0 && REG_PROMO >= ACC_REGS + 64 + 24 && COMET_PROMO_W64;
  static constexpr bool SB = !W64 && (TIGHT || (!LOADALL && COMET_PROMO_SB && REG_PROMO < ACC_REGS + 2 * 32 + 24 &&
                             REG_PROMO >= ACC_REGS + 32 + 24 && COLS % 32 == 0));
  static constexpr int PB = TIGHT ? 16 : LOADALL ? COLS
                          : ((SB || (REG_PROMO >= ACC_REGS + 2 * 32 + 24 && COLS % 32 == 0)) ? 32 : 16);
  static constexpr int NACC_TMEM = 512 / BN >= 4 ? 4 : 512 / BN;   // accumulators TMEM holds
  // NSUB = 2: each K-block is issued as two N = BN/2 sub-MMAs, one per promotion warpgroup, each
  // with its own ready / full barriers and issuing thread, so promotion of one half overlaps the
  // other half's MMAs and the accumulator ring is four half-units deep (BN = 256, NPW = 2).
  static constexpr int NSUB = (COMET_NSUB == 2 && NPW == 2 && BN / 2 >= 128) ? 2 : 1;
  // S pipeline slots, each holding one K-block's activation tile, packed and widened weights;
  // the scale ring has S + NACC slots (reuse is implied by the slot-free barrier, see below).
  // output staging for the TMA-store epilogue: per promotion WG two [128 rows][64 B] buffers
  // staging buffers per promotion WG: COMET_NSTAGE when the pipeline keeps >= 4 slots, else 2
  // shared-memory budget of the pipeline; COMET_N256_SMEM_KB overrides it for the 256-wide pair
  // tile alone (the pipeline-depth ablation: 160 -> S = 3)
  static constexpr int BUDGET_KB = (BN == 256 && CG == 2) ? COMET_N256_SMEM_KB : COMET_SMEM_BUDGET_KB;
  static constexpr int NSTAGE = (BUDGET_KB * 1024 - NPW * COMET_NSTAGE * 8192) / (SLOT_BYTES + BM * 4) >= 4
                                    ? COMET_NSTAGE : 2;
  static constexpr int STAGE_BYTES = NPW * NSTAGE * 8192;
  static constexpr int S_RAW = (BUDGET_KB * 1024 - STAGE_BYTES) / (SLOT_BYTES + BM * 4);
  // S must be even when two widen groups or two MMA issuers take alternate K-blocks: a waiter
  // that sees only every other K-block must see every phase of each slot it waits on (parity
  // waits cannot tell phase p from p + 2).  With an odd S a role could pass the wait for
  // K-block j + 2S on the completed phase of K-block j and read a slot still being filled
  // (tools/stress_gemm.py: intermittent launch failures of the 192-wide single-CTA tiles, S = 3).
  // An odd S >= 5 drops to S - 1; S = 3 keeps its depth with one widen group and one issuer.
  static constexpr int S_CAP = S_RAW > 8 ? 8 : S_RAW;
  static constexpr int S = (S_CAP % 2 == 1 && S_CAP >= 5) ? S_CAP - 1 : S_CAP;
  static constexpr int ISSUERS = S % 2 == 0 ? COMET_ISSUERS : 1;   // MMA issuing threads
  static_assert(S % 2 == 0 || NWG_ == 1, "alternating widen groups need an even slot count");
  // accumulators in TMEM; fewer than the slots (the promotion's release of K-block kb + NACC
  // lands on the mma_ready barrier of slot (kb + NACC) % S)
  static constexpr int NACC = NACC_TMEM < S ? NACC_TMEM : S - 1;
  static constexpr int SS = S + NACC;
  static constexpr int PRODUCERS = (COMET_PRODUCERS == 2 && S % 2 == 0 && SS % 2 == 0) ? 2 : 1;
  // [slots][output staging][scale ring SS x BM][w_scales 2 x BN][barriers][tmem][tags]
  // GS (NEXT-3 group-wise weight scales): per scale-ring slot also the K-block's weight scales
  // s_w[b][n0 .. n0+BN) (f32) and the tile rows' code sums qsum[b][m] (int16)
  static constexpr int GS_BYTES = GS_ ? SS * (BN * 4 + BM * 2) : 0;
  static constexpr int SMEM_DATA = S * SLOT_BYTES + STAGE_BYTES + SS * BM * 4 + 2 * BN * 4 + GS_BYTES;
  static constexpr int N_BARS = 2 * S + NSUB * S + NSUB * NACC;
  static constexpr int SMEM_BYTES = 1024 + SMEM_DATA + N_BARS * 8 + 16 + kMaxBlocks;
  static_assert(S >= 3, "pipeline depth");
  static_assert(SMEM_BYTES <= 232448, "shared memory per CTA");
  static_assert(S >= NACC + 1, "mma_ready ring must outlast the accumulator ring");
  static_assert(NACC % 2 == 0 || true, "");
  static_assert(NACC * BN <= 512, "TMEM budget");
  static_assert(COLS % 16 == 0, "promotion batches");
  static_assert(THREADS <= 1024, "threads per CTA");
  static_assert(REG_PROMO >= NEED, "promotion registers");
  static_assert(!(DEBUG_ && NSUB == 2), "debug kernels use whole-tile MMAs");
};

// Synchronisation (every role waits on exactly ONE mbarrier per K-block; a satisfied
// try_wait still costs ~180 clk on B200, see profiles/r01/probe_sync.json):
//   full[s]       TMA (activations, packed weights, scales) -> widen          [local]
//   slot_free[s]  MMA completion (multicast) + 4 local widen warps (packed W read) -> producer
//   mma_ready[s]  widen done for K-block kb (4 warps per CTA) + promotion done for K-block
//                 kb - NACC (8 warps per CTA, frees the accumulator kb reuses) -> MMA [even CTA]
//   acc_full[a]   MMA completion (multicast) -> promotion
// Implied orders: widen(kb) may overwrite widened slot s because the producer issued full[s] for
// kb only after slot_free[s] for kb - S; the scales of kb have landed when acc_full(kb) fires
// (MMA(kb) waited mma_ready(kb) which waited widen(kb) which waited full[s]); the producer may
// reuse scale slot kb % (S+NACC) because slot_free(kb-S) => MMA(kb-S) => promotion(kb-S-NACC).
template <int BN, int CG, int NPW, int NWG, int DEBUG, bool RS = false, bool GS = false>
__global__ void __launch_bounds__(CfgN<BN, CG, NPW, NWG, DEBUG, GS>::THREADS, 1) k_w4ax_n(const __grid_constant__ GemmParams P) {
  using C = CfgN<BN, CG, NPW, NWG, DEBUG, GS>;
  constexpr int kThreadsN = C::THREADS;
  constexpr int kPromoWarp0 = 4 + 4 * NWG;              // first promotion warp
  constexpr int S = C::S;
  constexpr int SS = C::SS;
  constexpr int NACC = C::NACC;
  constexpr int BM = C::BM;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  // slot s: [X: BM x 128 B][B: WROWS x 128 B][Wp: WROWS x 64 B]  (X and B 1024-aligned)
  auto sX = [&](int s) { return smem + s * C::SLOT_BYTES; };
  auto sB = [&](int s) { return smem + s * C::SLOT_BYTES + C::X_BYTES; };
  auto sWp = [&](int s) { return smem + s * C::SLOT_BYTES + C::X_BYTES + C::B_BYTES; };
  uint8_t* sY = smem + S * C::SLOT_BYTES;                                       // [NPW][2][8 KB]
  float* sS = reinterpret_cast<float*>(sY + C::STAGE_BYTES);                     // [SS][BM]
  float* sWs = sS + SS * BM;                                                     // [2][BN]
  float* sG = sWs + 2 * BN;                                                      // GS: [SS][BN]
  int16_t* sQ = reinterpret_cast<int16_t*>(sG + (GS ? SS * BN : 0));             // GS: [SS][BM]
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::SMEM_DATA);
  uint64_t* full = bars;                     // [S]
  uint64_t* slot_free = full + S;            // [S]
  uint64_t* mma_ready = slot_free + S;       // [NSUB][S]   (used in the even CTA)
  uint64_t* acc_full = mma_ready + C::NSUB * S;   // [NSUB][NACC]
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
  constexpr int NPROMO_WARPS = 4 * C::NPW;
  constexpr int NSUB = C::NSUB;
  // per sub-MMA: one widen group + the promotion warps that fold that sub-accumulator
  constexpr uint32_t kReadyCount = 4 * CG + (NPROMO_WARPS / NSUB) * CG;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&P.map_x);
    tma_prefetch(&P.map_w);
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&slot_free[i], NSUB + 4);        // MMA commit(s) + 4 widen warps
      for (int h = 0; h < NSUB; ++h) mbar_init(&mma_ready[h * S + i], kReadyCount);
    }
    for (int i = 0; i < NSUB * NACC; ++i) mbar_init(&acc_full[i], 1);
    // the first NACC K-blocks have no promotion predecessor
    for (int h = 0; h < NSUB; ++h)
      for (int i = 0; i < NACC; ++i) mbar_arrive_count(&mma_ready[h * S + i], (NPROMO_WARPS / NSUB) * CG);
    fence_mbar_init();
  }
  if (warp == 2) {
    if (CG == 2) { tmem_alloc_cg2<512>(tmem_holder); tmem_relinquish_cg2(); }
    else { tmem_alloc<512>(tmem_holder); tmem_relinquish(); }
  }
  for (int i = threadIdx.x; i < nb; i += kThreadsN) s_tags[i] = P.tags.get(i) ? 1 : 0;
  tc_fence_before();
  __syncthreads();
  if (CG == 2) cluster_sync();                 // peer barriers initialised before remote arrives
  tc_fence_after();
  const uint32_t tbase = *tmem_holder;
  // the even CTA's mma_ready barriers (shared::cluster addresses), arrived on by both CTAs
  const uint32_t ready_lead = CG == 2 ? mapa_shared(smem_u32(mma_ready), 0) : smem_u32(mma_ready);

  if (warp < 4) {
    setmaxnreg_dec<C::REG_LOW>();
    if ((warp == 0 || (C::PRODUCERS == 2 && warp == 2)) && lane == 0) {
      // ------------------------------------------------------------------ TMA producer(s)
      // TMA loads issued by one warp complete one after another (~1000 clk each under load,
      // profiles/r01/probe_stream.txt), so two warps (0 and 2) issue alternate K-blocks.  Each
      // producer only reuses its own slots (S even), so it observes every phase it waits on.
      const int par = warp == 0 ? 0 : 1;
      int j = 0, tr = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = load_item(P, it, debug);
        const int n_tile = w.tile / P.n_m_tiles, m_tile = w.tile % P.n_m_tiles;
        const int m0 = m_tile * (BM * CG) + BM * rank, n0 = n_tile * BN + C::WROWS * rank;
        const uint32_t sbytes = (m0 < P.Mp && !(COMET_STUB & 4)) ? (uint32_t)(min((int64_t)BM, P.Mp - m0) * 4) : 0u;
        const int64_t ng0 = (int64_t)n_tile * BN;              // GS: the whole tile's columns
        const uint32_t gbytes = GS ? (uint32_t)(min((int64_t)BN, P.N - ng0) * 4) : 0u;
        const uint32_t qbytes = GS ? sbytes / 2 : 0u;
        for (int kb = w.kb_begin; kb < w.kb_end; ++kb, ++j) {
          if (C::PRODUCERS == 2 && (j & 1) != par) continue;
          const int s = j % S, sc = j % SS;
          const uint32_t ph = (uint32_t)(j / S) & 1u;
          if (par == 0) trace_ev(P, 14, tr);
          mbar_wait(&slot_free[s], ph ^ 1);
          if (diag_ablate(P) & 32) {                       // diagnostic: no global loads
            mbar_arrive(&full[s]);
          } else {
            mbar_arrive_expect_tx(&full[s], C::X_BYTES + (COMET_PREWIDENED_UB ? C::B_BYTES : C::WP_BYTES) + sbytes + gbytes + qbytes);
            const uint8_t* src = reinterpret_cast<const uint8_t*>(P.scales) + ((kb * 7 + m0 / 128) % 32) * 24576;
            if (COMET_ABLATE_TMA2D & 1) bulk_load(sX(s), src, C::X_BYTES, &full[s]);
            else tma_load_2d(sX(s), &P.map_x, &full[s], kb * 128, m0);
            if (COMET_PREWIDENED_UB) {
              // the B half arrives as 128 rows x 128 B (an 8-bit weight tile's shape and bytes; the
              // values are the activation plane's -- timing only) straight into the MMA operand slot
              const int rb = (int)((n0 % (P.Mp > 256 ? P.Mp - 128 : 128)) & ~127);
              tma_load_2d(sB(s), &P.map_x, &full[s], kb * 128, rb);
            } else if (COMET_ABLATE_TMA2D & 2) {
              bulk_load(sWp(s), src + C::X_BYTES, C::WP_BYTES, &full[s]);
            } else {
              tma_load_4d(sWp(s), &P.map_w, &full[s], 0, 0, kb, n0 / kWTileRows);   // WROWS rows of K-block kb
            }
            if (sbytes) bulk_load(sS + sc * BM, P.scales + (int64_t)kb * P.Mp + m0, sbytes, &full[s]);
            if (GS) {
              bulk_load(sG + sc * BN, P.w_scales + (int64_t)kb * P.N + ng0, gbytes, &full[s]);
              if (qbytes) bulk_load(sQ + sc * BM, P.qsum + (int64_t)kb * P.Mp + m0, qbytes, &full[s]);
            }
          }
          if (par == 0) trace_ev(P, 0, tr++);
        }
      }
    } else if ((warp == 1 || (C::ISSUERS == 2 && warp == 3)) && rank == 0 && COMET_N_UNIFORM_MMA) {
      // ------------------------------------------------------------------ MMA issuers
      // Same schedule as below, but the whole warp runs the loop with warp-uniform operands
      // (shuffled from lane 0) so the MMA operands stay in uniform registers and one elected
      // lane issues the four MMAs back to back (no per-MMA R2UR waterfall).
      const int parity = warp == 1 ? 0 : 1;
      const int h = NSUB == 2 ? parity : 0;
      constexpr int NMMA = BN / NSUB;
      const uint32_t id_f8 = idesc_f8f6f4_e4m3(BM * CG, NMMA);
      const uint32_t id_i8 = idesc_i8(BM * CG, NMMA);
      const uint32_t tb = __shfl_sync(0xffffffffu, tbase, 0);
      const uint32_t sx0 = __shfl_sync(0xffffffffu, smem_u32(sX(0)), 0);
      int j = 0, tr = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = load_item(P, it, debug);
        const int kb_begin = __shfl_sync(0xffffffffu, w.kb_begin, 0);
        const int kb_end = __shfl_sync(0xffffffffu, w.kb_end, 0);
        for (int kb = kb_begin; kb < kb_end; ++kb, ++j) {
          if (NSUB == 1 && C::ISSUERS == 2 && (j & 1) != parity) continue;
          const int s = j % S, accb = j % NACC;
          const uint32_t ph = (uint32_t)(j / S) & 1u;
          if (lane == 0) trace_ev(P, parity ? 13 : 1, tr);
          if (COMET_MMA_WAIT_PLAIN) {
            // plain try_wait (no suspend hint); hang guard by iteration count, never read on the
            // fast path (each try_wait suspends for a hardware window, so 2^28 of them is seconds)
            uint32_t n = 0;
            while (!mbar_try_wait(smem_u32(&mma_ready[h * S + s]), ph))
              if (++n == (1u << 28)) __trap();
          }
          else if (COMET_SPIN_MMA) mbar_wait_spin(&mma_ready[h * S + s], ph); else mbar_wait(&mma_ready[h * S + s], ph);
          if (lane == 0) trace_ev(P, parity ? 11 : 3, tr);
          tc_fence_after();
          const uint32_t d = tb + accb * BN + h * NMMA;
          const uint32_t sa = sx0 + s * C::SLOT_BYTES;
          const uint32_t sbv = sa + C::X_BYTES + h * (C::WROWS / NSUB) * 128;
          const bool is8 = (COMET_STUB & 1) ? false : __shfl_sync(0xffffffffu, lds_u8(s_tags_a + kb), 0) != 0;
          // one elected thread issues the K-block's four MMAs AND its commits: tcgen05.commit
          // tracks the MMAs of the issuing thread only, so both must come from the same lane
          if (elect_one()) {
            if (diag_ablate(P) & 8) {
              // diagnostic: no MMA
            } else if (is8) {
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
              tc_commit_mc(&acc_full[h * NACC + accb], 3);
              tc_commit_mc(&slot_free[s], 3);
            } else {
              tc_commit(&acc_full[h * NACC + accb]);
              tc_commit(&slot_free[s]);
            }
          }
          __syncwarp();
          ++tr;
        }
      }
    } else if ((warp == 1 || (C::ISSUERS == 2 && warp == 3)) && lane == 0 && rank == 0 && !COMET_N_UNIFORM_MMA) {
      // ------------------------------------------------------------------ MMA issuers
      // Two issuing threads: warp 1 takes the even K-blocks of the CTA's sequence, warp 3 the
      // odd ones (different accumulators and slots), so one thread's barrier wait and commits
      // overlap the MMAs the other has queued.  tcgen05.commit tracks the issuing thread's own
      // MMAs, so each thread commits exactly the K-blocks it issued.
      // NSUB = 2: warp 1 issues sub-MMA 0 (accumulator columns [0, BN/2)) of every K-block and
      // warp 3 sub-MMA 1; each sub-MMA reads its half of every CTA's widened B rows.
      const int parity = warp == 1 ? 0 : 1;
      const int h = NSUB == 2 ? parity : 0;
      constexpr int NMMA = BN / NSUB;
      const uint32_t id_f8 = idesc_f8f6f4_e4m3(BM * CG, NMMA);
      const uint32_t id_i8 = idesc_i8(BM * CG, NMMA);
      int j = 0, tr = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = load_item(P, it, debug);
        for (int kb = w.kb_begin; kb < w.kb_end; ++kb, ++j) {
          if (NSUB == 1 && C::ISSUERS == 2 && (j & 1) != parity) continue;
          const int s = j % S, accb = j % NACC;
          const uint32_t ph = (uint32_t)(j / S) & 1u;
          trace_ev(P, parity ? 13 : 1, tr);
          if (COMET_SPIN_MMA) mbar_wait_spin(&mma_ready[h * S + s], ph); else mbar_wait(&mma_ready[h * S + s], ph);
          trace_ev(P, parity ? 11 : 3, tr++);
          tc_fence_after();
          const uint32_t d = tbase + accb * BN + h * NMMA;
          const uint32_t sa = smem_u32(sX(s));
          const uint32_t sbv = smem_u32(sB(s)) + h * (C::WROWS / NSUB) * 128;
          if (diag_ablate(P) & 8) {
            // diagnostic: no MMA
          } else if (lds_u8(s_tags_a + kb)) {
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
            tc_commit_mc(&acc_full[h * NACC + accb], 3);
            tc_commit_mc(&slot_free[s], 3);
          } else {
            tc_commit(&acc_full[h * NACC + accb]);
            tc_commit(&slot_free[s]);
          }
        }
      }
    }
  } else if (warp < kPromoWarp0) {
    setmaxnreg_dec<C::REG_WIDEN>();
    // -------------------------------------------------------------------- widen (W -> smem B)
    // The NWG widen warpgroups take K-blocks in turn; thread t of a group converts weight rows
    // t, t + 128, ... of its K-blocks.  INT4 block: byte = u (E4M3 u * 2^-9); INT8 block:
    // byte = 16 u - 128 = 16 w (s8), derived from the INT4-block form with one shift + xor.
    constexpr int RPT = (C::WROWS + 127) / 128;           // rows per thread
    const int grp = (warp - 4) >> 2;                      // K-blocks j with j % NWG == grp
    const int t = threadIdx.x - 128 - 128 * grp;
    int s = 0, tr = 0, j = 0;
    uint32_t ph = 0;
    for (int it = it_begin; it < it_end; ++it) {
      const WorkItem w = load_item(P, it, debug);
      for (int kb = w.kb_begin; kb < w.kb_end; ++kb, ++j) {
        if (NWG == 1 || j % NWG == grp) {
          const bool is8 = lds_u8(s_tags_a + kb) != 0;
          if (COMET_WIDEN_WAIT_PLAIN) { while (!mbar_try_wait(smem_u32(&full[s]), ph)) {} } else mbar_wait(&full[s], ph);
          if (warp == 4 && lane == 0) trace_ev(P, 5, tr);
          uint4 c[RPT][4];
#pragma unroll
          for (int i = 0; i < RPT; ++i) {
            const int row = t + 128 * i;
            if (row < C::WROWS && !(diag_ablate(P) & 64) && !COMET_PREWIDENED_UB) {   // 64: diagnostic, no widen loads
              const uint32_t src = smem_u32(sWp(s)) + row * 64;
              const int sw64 = (row >> 1) & 3;            // TMA 64-byte swizzle of the packed row
#pragma unroll
              for (int q4 = 0; q4 < 4; ++q4) c[i][q4] = lds128(src + ((q4 ^ sw64) << 4));
            }
          }
          __syncwarp();
          if (lane == 0) mbar_arrive(&slot_free[s]);     // packed weights of slot s consumed
#pragma unroll
          for (int i = 0; i < RPT; ++i) {
            const int row = t + 128 * i;
            if (row >= C::WROWS || (diag_ablate(P) & 4) || COMET_PREWIDENED_UB) break;
            const uint32_t dst = smem_u32(sB(s)) + row * 128;
            const int sw128 = row & 7;                    // UMMA 128-byte swizzle of the widened row
#pragma unroll
            for (int q4 = 0; q4 < 4; ++q4) {
              const uint32_t pw[4] = {c[i][q4].x, c[i][q4].y, c[i][q4].z, c[i][q4].w};
              uint32_t o[8];
#pragma unroll
              for (int k = 0; k < 4; ++k) widen_int4(pw[k], o[2 * k], o[2 * k + 1]);   // u[8g ..], u[8g+4 ..]
              if (is8) {                                  // warp-uniform: 5 % of blocks
#pragma unroll
                for (int k = 0; k < 8; ++k) o[k] = int4_to_int8(o[k]);
              }
              const int oc = 2 * q4;                      // logical 16-byte output chunk
              asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(dst + ((oc ^ sw128) << 4)),
                           "r"(o[0]), "r"(o[1]), "r"(o[2]), "r"(o[3]) : "memory");
              asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(dst + (((oc + 1) ^ sw128) << 4)),
                           "r"(o[4]), "r"(o[5]), "r"(o[6]), "r"(o[7]) : "memory");
            }
          }
          if (warp == 4 && lane == 0) trace_ev(P, 2, tr);
          fence_proxy_async_smem();                       // generic-proxy stores -> tensor core
          __syncwarp();
          if (lane == 0)
            for (int h = 0; h < NSUB; ++h) mbar_arrive_cluster(ready_lead + (h * S + s) * 8);
          if (warp == 4 && lane == 0) trace_ev(P, 4, tr);
          ++tr;
        }
        if (++s == S) { s = 0; ph ^= 1; }
      }
    }
  } else {
    setmaxnreg_inc<C::REG_PROMO>();
    // -------------------------------------------------------------------- promotion + epilogue
    const int wg = (warp - kPromoWarp0) >> 2;
    const int q = warp & 3;
    const int r = q * 32 + lane;                          // TMEM lane = token row within the tile
    const uint32_t lane_addr = (uint32_t)(q * 32) << 16;
    constexpr int COLS = C::COLS;
    const int col0 = wg * COLS;
    const int ptid = threadIdx.x - kPromoWarp0 * 32;
    const uint32_t s_scale_r = smem_u32(sS) + 4u * r;     // this row's scale in ring slot 0
    const uint32_t t_cols = tbase + col0 + lane_addr;     // this warp's columns in accumulator 0
    const int sub = NSUB == 2 ? wg : 0;                   // the sub-MMA whose columns this WG folds
    const uint32_t ready_rel = ready_lead + sub * S * 8;  // its mma_ready ring (even CTA)
    int accb = 0, sc = 0, rs = NACC % S, tr = 0;           // rs: mma_ready slot of kb + NACC
    uint32_t accph = 0;
    int tpar = 0;                                         // w_scales buffer of the current tile
    uint32_t ych = 0;                                     // output chunks this WG has staged
    // Accumulator column c of this WG -> weight row n of the tile (see the epilogue)
    constexpr int RUNS = (CG == 2 && NSUB == 2) ? 2 : 1;
    constexpr int RUN = COLS / RUNS;
    auto col_n = [&](int wgi, int c) -> int {             // offset from n0 (tile's first weight)
      return RUNS == 2 ? (c / RUN) * C::WROWS + wgi * RUN + (c % RUN) : wgi * COLS + c;
    };
    WorkItem wn = it_begin < it_end ? load_item(P, it_begin, debug) : WorkItem{};
    for (int it = it_begin; it < it_end; ++it) {
      const WorkItem w = wn;
      if (it + 1 < it_end) wn = load_item(P, it + 1, debug);   // in flight during this tile
      const int tp = tpar;                                // w_scales buffer of this tile
      tpar ^= 1;
      const int n_tile = w.tile / P.n_m_tiles, m_tile = w.tile % P.n_m_tiles;
      const int m0 = m_tile * (BM * CG) + BM * rank, n0 = n_tile * BN;
      const int64_t m = m0 + r;
      const bool owner = (w.flags & 2) != 0;
      const bool split = (w.flags & 1) != 0;
      // -corr * 2^-9 (offset-binary weight correction, owner segment only); loaded now, used
      // in the epilogue, so the load latency is off the K-loop's critical path
      // (GS: the offset term is removed per block instead, and there is no per-channel s_w)
      const float corr_raw = (!GS && owner && m < P.Mp) ? ldg_nc_f32(P.corr + m) : 0.f;
      // this tile's per-output-channel weight scales: loaded into registers now, written to
      // shared memory after the K-loop (read in the epilogue), so the global-load latency never
      // stalls the start of the tile's promotion
      constexpr int NWS = (BN + 128 * C::NPW - 1) / (128 * C::NPW);
      float wsv[NWS];
      if (!DEBUG) {
#pragma unroll
        for (int k = 0; k < NWS; ++k) {
          const int i = ptid + k * 128 * C::NPW;
          wsv[k] = 0.f;
          if (i < BN) {
            const int wgi = i / COLS, c = i % COLS;
            const int64_t n = (int64_t)n0 + col_n(wgi, c);
            if (n < P.N) wsv[k] = GS ? 1.f : __ldg(P.w_scales + n);
          }
        }
      }
      float acc[COLS];
      int32_t dacc[DEBUG ? COLS : 1];
#pragma unroll
      for (int c = 0; c < COLS; ++c) {
        acc[c] = 0.f;
        if (DEBUG) dacc[c] = 0;
      }
      for (int kb = w.kb_begin; kb < w.kb_end; ++kb) {
        const bool is8 = (COMET_STUB & 66) ? false : lds_u8(s_tags_a + kb) != 0;
        int qs = 0;
        if (DEBUG && !is8 && m < P.Mp) qs = P.qsum[(int64_t)kb * P.Mp + m];
        if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 12, tr);
        // Plain try_wait loop (no suspend-time hint, no timer): the hinted, timer-guarded wait
        // made the wake-up path slower AND kept ptxas from scheduling the post-wait address math
        // in the wait's shadow (3 % of the prefill GEMM, tools/gpu_pre_variants.sh).  A hang
        // here is still caught: acc_full(kb) completes unless MMA(kb) was never issued, and the
        // MMA issuer's own mma_ready wait is guarded (its trap aborts the launch).
        if (COMET_PROMO_WAIT_PLAIN) { while (!mbar_try_wait(smem_u32(&acc_full[sub * NACC + accb]), accph)) {} }
        else if (COMET_SPIN_PROMO) mbar_wait_spin(&acc_full[sub * NACC + accb], accph); else mbar_wait(&acc_full[sub * NACC + accb], accph);
        if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 6, tr);
        tc_fence_after();
        if (diag_ablate(P) & 16) {                              // diagnostic: no promotion work
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive_cluster(ready_rel + rs * 8);
          if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 7, tr);
          ++tr;
          if (++accb == NACC) { accb = 0; accph ^= 1; }
          if (++sc == SS) sc = 0;
          if (++rs == S) rs = 0;
          continue;
        }
        const uint32_t taddr = t_cols + accb * BN;
        // LOADALL: one load of all COLS columns, release, then fold.  Otherwise software-
        // pipelined over PB-column batches: the load of batch b+1 is in flight while batch b is
        // folded in; the accumulator is released once the last load has landed.
        constexpr int PB = C::PB;                         // columns per TMEM load batch
        constexpr int NB_ = COLS / PB;
        // the row's activation scale of this K-block (shared-memory ring slot sc), times 2^-13 for
        // an INT8 block (acc = 16 sum x w)
        auto row_scale = [&]() -> float {
          float s = 1.0f;
          if (!(COMET_STUB & 34)) asm volatile("ld.shared.f32 %0, [%1];" : "=f"(s) : "r"(s_scale_r + 4u * BM * sc));
          return is8 ? s * 1.220703125e-04f : s;
        };
        if constexpr (C::W64 && GS) {
          const float s = row_scale();
          const float2 s2 = make_float2(s, s);
          // GS (NEXT-3, reading R18): per column n the K-block's weight scale s_w[b][n] joins
          // the row's s_a[m,b], and an INT4 block's offset-binary term 2^-6 qsum[b][m] is removed
          // per block: acc += (s_a v - s_a 2^-6 qsum) * s_w[b][n] -- the bracket is one FFMA2
          // with row scalars, the s_w product a second: two packed operations per two columns
          float qc = 0.f;
          if (GS && !is8) qc = -(float)sQ[sc * BM + r] * 0.015625f * s;   // -s_a 2^-6 qsum
          const float2 qc2 = make_float2(qc, qc);
          const float* gsw = sG + sc * BN + col0;
          if constexpr (GS) {
#pragma unroll
            for (int b = 0; b < COLS / 64; ++b) {
              uint32_t v[64];
              tmem_ld_32x32b<64>(taddr + b * 64, v);
              tmem_wait_ld();
              if (b + 1 == COLS / 64) {
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive_cluster(ready_rel + rs * 8);
              }
#pragma unroll
              for (int c = 0; c < 64; c += 4) {
                const int a = b * 64 + c;
                const float4 w4 = *reinterpret_cast<const float4*>(gsw + a);   // broadcast smem load
                float2 x0, x1;
                if (is8) {
                  x0 = i2f2_exact(v[c], v[c + 1]);
                  x1 = i2f2_exact(v[c + 2], v[c + 3]);
                } else {
                  x0 = make_float2(__uint_as_float(v[c]), __uint_as_float(v[c + 1]));
                  x1 = make_float2(__uint_as_float(v[c + 2]), __uint_as_float(v[c + 3]));
                }
                const float2 u0 = ffma2(x0, s2, qc2), u1 = ffma2(x1, s2, qc2);   // s_a v - s_a 2^-6 qsum
                const float2 y0 = ffma2(u0, make_float2(w4.x, w4.y), make_float2(acc[a], acc[a + 1]));
                const float2 y1 = ffma2(u1, make_float2(w4.z, w4.w), make_float2(acc[a + 2], acc[a + 3]));
                acc[a] = y0.x; acc[a + 1] = y0.y; acc[a + 2] = y1.x; acc[a + 3] = y1.y;
              }
            }
            ++tr;
            if (++accb == NACC) { accb = 0; accph ^= 1; }
            if (++sc == SS) sc = 0;
            if (++rs == S) rs = 0;
            continue;
          }
        }
        if constexpr (C::W64 && !GS) {
          float2 s2;
#pragma unroll
          for (int b = 0; b < COLS / 64; ++b) {
            uint32_t v[64];
            if (COMET_LDTM_X64) tmem_ld_32x32b_x64(taddr + b * 64, v); else tmem_ld_32x32b<64>(taddr + b * 64, v);
            if (b == 0) {
              const float s = row_scale();
              s2 = make_float2(s, s);
            }
            tmem_wait_ld();
            if (b == 0 && threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 9, tr);
            if (b + 1 == COLS / 64) {
              // every accumulator column of this thread is in registers: release the buffer
              tc_fence_before();
              __syncwarp();
              if (lane == 0) mbar_arrive_cluster(ready_rel + rs * 8);
              if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 10, tr);
            }
            if (is8) {                                    // warp-uniform (5 % of blocks)
#pragma unroll
              for (int c = 0; c < 64; c += 2) {
                const int a = b * 64 + c;
                const float2 y = ffma2(i2f2_exact(v[c], v[c + 1]), s2, make_float2(acc[a], acc[a + 1]));
                acc[a] = y.x;
                acc[a + 1] = y.y;
              }
            } else {
#pragma unroll
              for (int c = 0; c < 64; c += 2) {
                const int a = b * 64 + c;
                if (COMET_PROMO_SCALAR) {
                  acc[a] = __fmaf_rn(__uint_as_float(v[c]), s2.x, acc[a]);
                  acc[a + 1] = __fmaf_rn(__uint_as_float(v[c + 1]), s2.y, acc[a + 1]);
                } else {
                  const float2 y = ffma2(make_float2(__uint_as_float(v[c]), __uint_as_float(v[c + 1])), s2,
                                         make_float2(acc[a], acc[a + 1]));
                  acc[a] = y.x;
                  acc[a + 1] = y.y;
                }
              }
            }
          }
          if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 7, tr);
          ++tr;
          if (++accb == NACC) { accb = 0; accph ^= 1; }
          if (++sc == SS) sc = 0;
          if (++rs == S) rs = 0;
          continue;
        }
        if constexpr (C::SB) {
          // single-buffered batches: load, wait, fold; release after the last load landed
          float s;
          asm volatile("ld.shared.f32 %0, [%1];" : "=f"(s) : "r"(s_scale_r + 4u * BM * sc));
          if (is8) s *= 1.220703125e-04f;
          const float2 s2 = make_float2(s, s);
#pragma unroll
          for (int b = 0; b < NB_; ++b) {
            uint32_t v[PB];
            tmem_ld_32x32b<PB>(taddr + b * PB, v);
            tmem_wait_ld();
            if (b == 0 && threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 9, tr);
            if (b + 1 == NB_) {
              tc_fence_before();
              __syncwarp();
              if (lane == 0) mbar_arrive_cluster(ready_rel + rs * 8);
              if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 10, tr);
            }
            if (is8) {
#pragma unroll
              for (int c = 0; c < PB; c += 2) {
              const float2 f = i2f2_exact(v[c], v[c + 1]);
              v[c] = __float_as_uint(f.x);
              v[c + 1] = __float_as_uint(f.y);
            }
            }
#pragma unroll
            for (int c = 0; c < PB; c += 2) {
              const int a = b * PB + c;
              float2 y = ffma2(make_float2(__uint_as_float(v[c]), __uint_as_float(v[c + 1])), s2,
                               make_float2(acc[a], acc[a + 1]));
              acc[a] = y.x;
              acc[a + 1] = y.y;
            }
          }
          if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 7, tr);
          ++tr;
          if (++accb == NACC) { accb = 0; accph ^= 1; }
          if (++sc == SS) sc = 0;
          if (++rs == S) rs = 0;
          continue;
        }
        uint32_t vb[NB_ > 1 ? 2 : 1][PB];
        tmem_ld_32x32b<PB>(taddr, vb[0]);
        if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 8, tr);
        float s;
        asm volatile("ld.shared.f32 %0, [%1];" : "=f"(s) : "r"(s_scale_r + 4u * BM * sc));
        if (is8) s *= 1.220703125e-04f;                   // 2^-13: INT8 block acc = 16 sum x w
        const float2 s2 = make_float2(s, s);
        tmem_wait_ld();
        if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 9, tr);
        if (NB_ == 1) {
          // every accumulator column of this thread is in registers: release the TMEM buffer
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive_cluster(ready_rel + rs * 8);
        }
#pragma unroll
        for (int b = 0; b < NB_; ++b) {
          uint32_t* v = vb[NB_ > 1 ? (b & 1) : 0];
          if (b + 1 < NB_) tmem_ld_32x32b<PB>(taddr + (b + 1) * PB, vb[NB_ > 1 ? ((b + 1) & 1) : 0]);
          if (DEBUG) {
#pragma unroll
            for (int c = 0; c < PB; ++c) {
              const int32_t ab = is8 ? (((int32_t)v[c]) >> 4) : ((int32_t)(__uint_as_float(v[c]) * 512.f) - 8 * qs);
              dacc[b * PB + c] += ab;
              if (DEBUG == 2 && m < P.M && n0 + col0 + b * PB + c < P.N)
                P.dbg_blocks[((int64_t)kb * P.M + m) * P.N + n0 + col0 + b * PB + c] = ab;
            }
          }
          if (is8) {
#pragma unroll
            for (int c = 0; c < PB; c += 2) {
              const float2 f = i2f2_exact(v[c], v[c + 1]);
              v[c] = __float_as_uint(f.x);
              v[c + 1] = __float_as_uint(f.y);
            }
          }
#pragma unroll
          for (int c = 0; c < PB; c += 2) {
            const int a = b * PB + c;
            float2 y = ffma2(make_float2(__uint_as_float(v[c]), __uint_as_float(v[c + 1])), s2,
                             make_float2(acc[a], acc[a + 1]));
            acc[a] = y.x;
            acc[a + 1] = y.y;
          }
          if (b + 1 < NB_) {
            tmem_wait_ld();
            if (b + 2 == NB_) {
              // every accumulator column of this thread is now in registers: release the TMEM
              // buffer (the MMA for kb + NACC may start) before the last batch's math
              tc_fence_before();
              __syncwarp();
              if (lane == 0) mbar_arrive_cluster(ready_rel + rs * 8);
              if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 10, tr);
            }
          }
        }
        if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 7, tr);
        ++tr;
        if (++accb == NACC) { accb = 0; accph ^= 1; }
        if (++sc == SS) sc = 0;
        if (++rs == S) rs = 0;
      }
      if (!DEBUG) {
#pragma unroll
        for (int k = 0; k < NWS; ++k) {
          const int i = ptid + k * 128 * C::NPW;
          if (i < BN) sWs[tp * BN + i] = wsv[k] * 512.f;   // s_w * 2^9 (exact scaling)
        }
      }
      // ---------------------------------------------------------------- epilogue
      const float init = (COMET_STUB & 128) ? 0.f : -corr_raw * 0.001953125f;   // -corr * 2^-9 (0 for GS / non-owners)
      if (split) {
        const int seg = (w.flags >> 8) & 0xFF;
        const int nseg = (w.flags >> 16) & 0xFF;
        // partial tile: float4 (a/4, ptid) at [(a/4) * NT + ptid] -- a warp's stores are contiguous
        const int64_t part_tile = (int64_t)BM * BN;        // = NT promotion threads * COLS floats
        constexpr int NT = 128 * C::NPW;
        if (!owner) {
          float4* dst = reinterpret_cast<float4*>(
              P.ws_part + (((int64_t)w.fix * (P.max_seg - 1) + (seg - 1)) * CG + rank) * part_tile) + ptid;
#pragma unroll
          for (int a = 0; a < COLS; a += 4) dst[(a / 4) * NT] = make_float4(acc[a], acc[a + 1], acc[a + 2], acc[a + 3]);
          __threadfence();
          named_bar_sync(1, 128 * C::NPW);
          if (threadIdx.x == kPromoWarp0 * 32) st_release_gpu(P.ws_flags + ((int64_t)w.fix * P.max_seg + seg) * CG + rank, P.epoch);
          continue;
        }
        if (threadIdx.x == kPromoWarp0 * 32) {
          for (int sgi = 1; sgi < nseg; ++sgi) {
            const uint32_t* f = P.ws_flags + ((int64_t)w.fix * P.max_seg + sgi) * CG + rank;
            uint64_t t0g = globaltimer_ns();
            while (ld_acquire_gpu(f) != P.epoch) {
              if (globaltimer_ns() - t0g > COMET_MBAR_TIMEOUT_NS) {
                __trap();
              }
            }
            *const_cast<uint32_t*>(f) = 0u;   // consumed: every launch leaves the flags zeroed
          }
        }
        named_bar_sync(1, 128 * C::NPW);
        for (int sgi = 1; sgi < nseg; ++sgi) {
          const float4* src = reinterpret_cast<const float4*>(
              P.ws_part + (((int64_t)w.fix * (P.max_seg - 1) + (sgi - 1)) * CG + rank) * part_tile) + ptid;
#pragma unroll
          for (int a = 0; a < COLS; a += 4) {
            float4 t4;
            asm volatile("ld.global.cg.v4.f32 {%0,%1,%2,%3}, [%4];"
                         : "=f"(t4.x), "=f"(t4.y), "=f"(t4.z), "=f"(t4.w) : "l"(src + (a / 4) * NT));
            acc[a] += t4.x; acc[a + 1] += t4.y; acc[a + 2] += t4.z; acc[a + 3] += t4.w;
          }
        }
      }
      if (DEBUG) {
        // Debug kernels: direct stores (plus the exact integer accumulators).
        if (m < P.M) {
          const int nbase = n0 + col0;
          if (nbase < P.N) {
            const int nvalid = (int)min((int64_t)COLS, (int64_t)P.N - nbase);
#pragma unroll
            for (int c = 0; c < COLS; ++c) {
              if (c >= nvalid) continue;
              const float f = (acc[c] + init) * __ldg(P.w_scales + nbase + c) * 512.f;
              if (P.ydt == COMET_F32) reinterpret_cast<float*>(P.y)[m * P.ldy + nbase + c] = f;
              else if (P.ydt == COMET_BF16) reinterpret_cast<__nv_bfloat16*>(P.y)[m * P.ldy + nbase + c] = __float2bfloat16_rn(f);
              else reinterpret_cast<__half*>(P.y)[m * P.ldy + nbase + c] = __float2half_rn(f);
              P.dbg_acc[m * P.N + nbase + c] = dacc[c];
            }
          }
        }
      } else if constexpr (RS) {
        // NEXT-2: the row-parallel layer's reduce-scatter fused into the epilogue (P:L373
        // "operator pipelining"): this rank's FP32 partial y_r = (acc - corr 2^-9) s_w 2^9 of row m
        // goes straight to the owner of row m over NVLink -- the transfer of tile t overlaps the
        // MMAs of tile t+1 -- and comet_rs_reduce sums the ranks' slots there in rank order.
        named_bar_sync(1, 128 * C::NPW);                  // this tile's w_scales are in smem
        const float* sw = sWs + tp * BN + wg * COLS;
        if (m < P.M) {
          const int owner = (int)(m / P.rs_ms);
          const int64_t ml = m - (int64_t)owner * P.rs_ms;
          float* dst = P.rs_dst[owner] + ((int64_t)P.rs_rank * P.rs_ms + ml) * P.N + n0;
#pragma unroll
          for (int c = 0; c < COLS; c += 4) {
            const int64_t nc = col_n(wg, c);              // 4 consecutive columns from here
            if (n0 + nc >= P.N) continue;
            const float4 v = make_float4((acc[c] + init) * sw[c], (acc[c + 1] + init) * sw[c + 1],
                                         (acc[c + 2] + init) * sw[c + 2], (acc[c + 3] + init) * sw[c + 3]);
            asm volatile("st.global.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(dst + nc), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w) : "memory");
          }
        }
      } else if (COMET_STUB & 8) {
        // timing experiment: no epilogue
      } else {
        // TMA-store epilogue.  y = (acc - corr 2^-9) * s_w * 512 (R7).  The
        // WG's COLS columns leave in chunks of 64 bytes per row (32 half / 16 float columns),
        // staged in a double-buffered, 64B-swizzled [128 rows][64 B] shared tile and written by
        // one TMA tensor store each (coalesced; rows >= M and columns >= N are clipped).
        if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 15, 4 * (it - it_begin));
        if (!(COMET_STUB & 256)) named_bar_sync(1, 128 * C::NPW);   // this tile's w_scales are in smem
        if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 15, 4 * (it - it_begin) + 1);
        const float* sw = sWs + tp * BN + wg * COLS;
        uint8_t* stage = sY + wg * C::NSTAGE * 8192;
        const uint32_t swz = (uint32_t)((r >> 1) & 3);
        const bool leader = (threadIdx.x & 127) == 0;     // thread 0 of the WG (row 0)
        // COMET_EPI_WARP: each warp stores its own 32 rows with its own TMA store (box 32 rows),
        // synchronising only within the warp; otherwise one store per warpgroup chunk.
        auto stage_and_store = [&](const uint32_t (&pk)[16], int ncol_off, int esz) {
          // caller: buffer (ych % NSTAGE) is free (see the wait below)
          const uint32_t rowa = smem_u32(stage + (ych % C::NSTAGE) * 8192) + r * 64;
          if (!(COMET_STUB & 1024)) {
#pragma unroll
            for (int k = 0; k < 4; ++k)
              asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(rowa + ((k ^ swz) << 4)),
                           "r"(pk[4 * k]), "r"(pk[4 * k + 1]), "r"(pk[4 * k + 2]), "r"(pk[4 * k + 3]) : "memory");
          } else {
            if ((pk[0] ^ pk[5] ^ pk[10] ^ pk[15]) == 0x12345678u) asm volatile("st.shared.u32 [%0], %1;" ::"r"(rowa), "r"(pk[1]) : "memory");
          }
          if (COMET_STUB & 512) { ++ych; return; }
          fence_proxy_async_smem();
          if (COMET_EPI_WARP) {
            __syncwarp();
            if (lane == 0) {
              tma_store_2d(&P.map_y, stage + (ych % C::NSTAGE) * 8192 + (warp & 3) * 32 * 64,
                           (n0 + col_n(wg, ncol_off)) * esz, m0 + (warp & 3) * 32);
              bulk_commit_group();
            }
          } else {
            named_bar_sync(2 + wg, 128);
            if (leader) {
              tma_store_2d(&P.map_y, stage + (ych % C::NSTAGE) * 8192, (n0 + col_n(wg, ncol_off)) * esz, m0);
              bulk_commit_group();
            }
          }
          ++ych;
        };
        auto wait_buffer = [&]() {                        // the store NSTAGE chunks ago has read its buffer
          if (COMET_EPI_WARP) {
            if (lane == 0) bulk_wait_group_read<C::NSTAGE - 1>();
            __syncwarp();
          } else {
            if (leader) bulk_wait_group_read<C::NSTAGE - 1>();
            named_bar_sync(2 + wg, 128);
          }
        };
        if (P.ydt == COMET_F32) {
#pragma unroll
          for (int q = 0; q < COLS / 16; ++q) {
            wait_buffer();
            uint32_t pk[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) pk[i] = __float_as_uint((acc[q * 16 + i] + init) * sw[q * 16 + i]);
            stage_and_store(pk, q * 16, 4);
          }
        } else {
          const bool bf = P.ydt == COMET_BF16;
#pragma unroll
          for (int q = 0; q < COLS / 32; ++q) {
            wait_buffer();
            uint32_t pk[16];
#pragma unroll
            for (int i = 0; i < 16; i += 2) {
              // y = (acc + init) s' = acc s' + init s'  (s' = s_w 2^9), as two FFMA2 pairs
              const int c = q * 32 + 2 * i;
              const float4 s4 = *reinterpret_cast<const float4*>(sw + c);
              const float2 y0 = ffma2(make_float2(acc[c], acc[c + 1]), make_float2(s4.x, s4.y),
                                      make_float2(init * s4.x, init * s4.y));
              const float2 y1 = ffma2(make_float2(acc[c + 2], acc[c + 3]), make_float2(s4.z, s4.w),
                                      make_float2(init * s4.z, init * s4.w));
              if (bf) {
                __nv_bfloat162 h0 = __floats2bfloat162_rn(y0.x, y0.y), h1 = __floats2bfloat162_rn(y1.x, y1.y);
                pk[i] = *reinterpret_cast<uint32_t*>(&h0);
                pk[i + 1] = *reinterpret_cast<uint32_t*>(&h1);
              } else {
                __half2 h0 = __floats2half2_rn(y0.x, y0.y), h1 = __floats2half2_rn(y1.x, y1.y);
                pk[i] = *reinterpret_cast<uint32_t*>(&h0);
                pk[i + 1] = *reinterpret_cast<uint32_t*>(&h1);
              }
            }
            stage_and_store(pk, q * 32, 2);
            if (q == 1 && threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 15, 4 * (it - it_begin) + 2);
          }
          if constexpr (COLS % 32 == 16) {
            // the last 16 columns (tile_w = 160: 80 per warpgroup) do not fill a 64-byte TMA
            // chunk: each thread stores its row's 32 bytes directly
            constexpr int c0 = COLS - 16;
            uint32_t pk[8];
#pragma unroll
            for (int i = 0; i < 8; i += 2) {
              const int c = c0 + 2 * i;
              const float4 s4 = *reinterpret_cast<const float4*>(sw + c);
              const float2 y0 = ffma2(make_float2(acc[c], acc[c + 1]), make_float2(s4.x, s4.y),
                                      make_float2(init * s4.x, init * s4.y));
              const float2 y1 = ffma2(make_float2(acc[c + 2], acc[c + 3]), make_float2(s4.z, s4.w),
                                      make_float2(init * s4.z, init * s4.w));
              if (bf) {
                __nv_bfloat162 h0 = __floats2bfloat162_rn(y0.x, y0.y), h1 = __floats2bfloat162_rn(y1.x, y1.y);
                pk[i] = *reinterpret_cast<uint32_t*>(&h0);
                pk[i + 1] = *reinterpret_cast<uint32_t*>(&h1);
              } else {
                __half2 h0 = __floats2half2_rn(y0.x, y0.y), h1 = __floats2half2_rn(y1.x, y1.y);
                pk[i] = *reinterpret_cast<uint32_t*>(&h0);
                pk[i + 1] = *reinterpret_cast<uint32_t*>(&h1);
              }
            }
            const int64_t n = (int64_t)n0 + col_n(wg, c0);
            if (m < P.M && n < P.N) {
              uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<uint16_t*>(P.y) + m * P.ldy + n);
              dst[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
              dst[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
            }
          }
        }
        if (threadIdx.x == kPromoWarp0 * 32) trace_ev(P, 15, 4 * (it - it_begin) + 3);
      }
    }
    if (!DEBUG && (COMET_EPI_WARP ? lane == 0 : (threadIdx.x & 127) == 0)) bulk_wait_group<0>();   // all output stores done
  }

  tc_fence_before();
  __syncthreads();
  if (CG == 2) cluster_sync();                 // the pair is done with each other's smem / TMEM
  if (warp == 2) {
    if (CG == 2) tmem_dealloc_cg2<512>(tbase); else tmem_dealloc<512>(tbase);
  }
}

template <int BN, int CG, int NPW, int NWG, int DEBUG, bool RS = false, bool GS = false>
cudaError_t launch_bn(const GemmParams& prm, int grid, cudaStream_t stream) {
  using C = CfgN<BN, CG, NPW, NWG, DEBUG, GS>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t ea = set_smem_attr(k_w4ax_n<BN, CG, NPW, NWG, DEBUG, RS, GS>, C::SMEM_BYTES, attr_done);
  if (ea != cudaSuccess) return ea;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(C::THREADS);
  cfg.dynamicSmemBytes = C::SMEM_BYTES;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CG;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k_w4ax_n<BN, CG, NPW, NWG, DEBUG, RS, GS>, prm);
}

// Persistent units (CTAs, or CTA pairs for CG = 2) of this kernel that can be resident at once.
template <int BN, int CG, int NPW, int NWG, int DEBUG>
int max_units_bn(int sms) {
  using C = CfgN<BN, CG, NPW, NWG, DEBUG>;
  auto kern = k_w4ax_n<BN, CG, NPW, NWG, DEBUG>;
  static std::atomic<uint64_t> attr_done{0};
  if (set_smem_attr(kern, C::SMEM_BYTES, attr_done) != cudaSuccess) return -1;
  if (CG == 1) {
    int b = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kern, C::THREADS, C::SMEM_BYTES) != cudaSuccess) return -1;
    return b * sms;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(CG * sms / CG));
  cfg.blockDim = dim3(C::THREADS);
  cfg.dynamicSmemBytes = C::SMEM_BYTES;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = CG;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, kern, &cfg) != cudaSuccess) return -1;
  return n;
}

}  // namespace

int stages_gemm_n(int bn, int cg) {
  if (cg == 2) {
    if (bn == 192) return CfgN<192, 2, 3, 2, 0>::S;
    if (bn == 160) return CfgN<160, 2, 2, 2, 0>::S;
    if (bn == 128) return CfgN<128, 2, 2, 2, 0>::S;
    return CfgN<256, 2, COMET_N256_NPW, COMET_N256_NWG, 0>::S;
  }
  if (bn == 192) return CfgN<192, 1, 3, 1, 0>::S;
  if (bn == 160) return CfgN<160, 1, 2, 1, 0>::S;
  return CfgN<128, 1, 2, 2, 0>::S;
}

int max_units_gemm_n(int bn, int cg, int sms) {
  if (cg == 2) {
    if (bn == 192) return max_units_bn<192, 2, 3, 2, 0>(sms);
    if (bn == 160) return max_units_bn<160, 2, 2, 2, 0>(sms);
    if (bn == 128) return max_units_bn<128, 2, 2, 2, 0>(sms);
    return max_units_bn<256, 2, COMET_N256_NPW, COMET_N256_NWG, 0>(sms);
  }
  if (bn == 192) return max_units_bn<192, 1, 3, 1, 0>(sms);
  if (bn == 160) return max_units_bn<160, 1, 2, 1, 0>(sms);
  return max_units_bn<128, 1, 2, 2, 0>(sms);
}

// bn = 128, 160, 192 or 256; 96 for the debug-accumulator kernels (they need the registers).
cudaError_t launch_gemm_n(const GemmParams& prm, int grid, int bn, int cg, int debug, cudaStream_t stream,
                          bool grouped) {
  if (grouped) {
    // NEXT-3 group-wise weight scales: the 256-wide pair kernel with the grouped promotion
    if (cg != 2 || bn != 256 || debug || prm.rs_world > 0) return cudaErrorInvalidValue;
    return launch_bn<256, 2, COMET_N256_NPW, COMET_N256_NWG, 0, false, true>(prm, grid, stream);
  }
  if (prm.rs_world > 0) {
    // NEXT-2 fused reduce-scatter: the 256-wide pair kernel with the peer-store epilogue
    if (cg != 2 || bn != 256 || debug) return cudaErrorInvalidValue;
    return launch_bn<256, 2, COMET_N256_NPW, COMET_N256_NWG, 0, true>(prm, grid, stream);
  }
  if (cg == 2) {
    if (debug == 2) return launch_bn<96, 2, 3, 2, 2>(prm, grid, stream);
    if (debug == 1) return launch_bn<96, 2, 3, 2, 1>(prm, grid, stream);
    if (bn == 192) return launch_bn<192, 2, 3, 2, 0>(prm, grid, stream);
    if (bn == 160) return launch_bn<160, 2, 2, 2, 0>(prm, grid, stream);
    if (bn == 128) return launch_bn<128, 2, 2, 2, 0>(prm, grid, stream);
    return launch_bn<256, 2, COMET_N256_NPW, COMET_N256_NWG, 0>(prm, grid, stream);
  }
  if (debug == 2) return launch_bn<96, 1, 3, 2, 2>(prm, grid, stream);
  if (debug == 1) return launch_bn<96, 1, 3, 2, 1>(prm, grid, stream);
  // S = 3 at these widths: one widen group, one issuer (see CfgN::S)
  if (bn == 192) return launch_bn<192, 1, 3, 1, 0>(prm, grid, stream);
  if (bn == 160) return launch_bn<160, 1, 2, 1, 0>(prm, grid, stream);
  if (bn == 128) return launch_bn<128, 1, 2, 2, 0>(prm, grid, stream);
  return cudaErrorInvalidValue;   // the single-CTA kernel has no 256-wide variant (planner rejects it)
}

}  // namespace gemm
}  // namespace comet
