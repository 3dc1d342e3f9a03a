// gemm.cu -- the W4Ax GEMM for decode-sized token counts on sm_100a (kernel 2, orientation 1),
// persistent, warp-specialised, HBM-streaming; plus the host-side launcher of both GEMM kernels.
//
//   Y[m, n] = s_w[n] * sum_b s_a[m,b] * acc_b[m,n]
//
// One CTA per SM walks the planner's work list (tile, K-block range).  An output
// tile is 128 weight rows (n) x NT tokens (m).  The MMA runs "transposed": the weight tile is
// the A operand (M = 128 rows, held in TENSOR MEMORY after widening), the activation tile is
// the B operand (N = NT tokens, TMA-staged in shared memory, 128-byte swizzle), so the tokens
// become the MMA N dimension and decode-sized M still fills an instruction.
//
// At decode sizes the kernel is a weight stream: the packed weights (N*K/2 bytes) dominate the
// traffic.  A pipeline stage therefore carries several K-blocks (KS): one 4D TMA box of the 128
// rows' KS K-blocks of packed weights (the row-tiled layout makes each 16-row tile's KS K-blocks
// one contiguous KS-KB run, include/comet.h), the K-blocks' activation codes and their scales.
//
// Roles (512 threads, 16 warps):
//   warp 0       TMA producer of the weight ring (lane 0).
//   warp 1       MMA issuer: per K-block 4 x tcgen05.mma (K = 32) into its own TMEM
//                accumulator; INT4 blocks use kind::f8f6f4 (E4M3), INT8 blocks kind::i8.
//   warp 2       TMEM allocator; TMA producer of the activation ring (lane 0): codes + scales.
//   warps 4-11   widen, two groups of 4 warps taking alternate stages: a packed INT4 weight row
//                -> 256 bytes in 3 instructions per 8 values (the B200 form of the paper's
//                location switch + zero extension), tcgen05.st into a TMEM A buffer.
//                INT4 block: byte = u = w+8, read by the FP8 tensor core as u * 2^-9 exactly.
//                INT8 block: byte = 16*w (s8).
//   warps 12-15  promotion ("dequant"): per K-block, tcgen05.ld the accumulator (thread =
//                weight row, columns = tokens) and fold it into FP32 registers with the block's
//                per-token scale (FFMA2); at the end of the tile the FP32 result is scaled by s_w
//                and stored (or, for a tile split across CTAs, exchanged through the stream-K
//                workspace in a fixed order).
//
// Exactness: INT4 block: acc = 2^-9 * sum_k x_k (w_k + 8) with every term an integer multiple
// of 2^-9 and |sum| < 2^14 -> exact in FP32 (checked bit-exactly against the oracle through the
// debug accumulators); the +8 offset is removed with corr[m] = 8 sum_b s_a qsum (kernel 1).
// INT8 block: acc = 16 * sum_k x_k w_k exactly in INT32.
#include <algorithm>
#include <cstdlib>
#include "gemm_common.cuh"
#include "fmpq.cuh"

// The pipeline roles' waits (promotion 1, MMA issuer 2, widen 4) are bare try_wait loops: ~2 %
// faster than the timer-guarded mbar_wait on every decode shape (tools/gpu_decb_variants.sh);
// even an iteration-count guard (COMET_DEC_GUARD) gave the gain back.  The two producers' waits
// keep the timer guard: a stalled pipeline stops releasing their ring slots, so their guarded
// waits trap; the unguarded window is a CTA's last ring-depth of stages, where every load has
// been issued and only a load that never completes could hang.
#ifndef COMET_DEC_PLAIN
#define COMET_DEC_PLAIN 7
#endif
#ifndef COMET_DEC_GUARD
#define COMET_DEC_GUARD 0   // which of them count iterations as a hang guard (experiment)
#endif
#define DEC_WAIT(bit, bar, ph)                                                                  \
  do {                                                                                          \
    if (COMET_DEC_PLAIN & COMET_DEC_GUARD & (bit)) {                                            \
      uint32_t n_ = 0;                                                                          \
      while (!mbar_try_wait(smem_u32(bar), (ph)))                                               \
        if (++n_ == (1u << 28)) __trap();                                                       \
    } else if (COMET_DEC_PLAIN & (bit)) {                                                       \
      while (!mbar_try_wait(smem_u32(bar), (ph))) {}                                            \
    } else {                                                                                    \
      mbar_wait((bar), (ph));                                                                   \
    }                                                                                           \
  } while (0)


namespace comet {
namespace gemm {
namespace {
#ifndef COMET_DEC_ABLATE
#define COMET_DEC_ABLATE 0      // timing experiments only (wrong results): bit 0 no MMAs, bit 1 no
#endif                          // TMEM stores of widened weights, bit 2 no accumulator loads,
                                // bit 3 no weight reads by the widen warps, bit 4 no activation loads

#ifndef COMET_DEC_NA
#define COMET_DEC_NA 2
#endif
#ifndef COMET_DEC_ST64
#define COMET_DEC_ST64 0    // 1: one 64-column TMEM store per widen warp and stage (KS = 4)
#endif
#ifndef COMET_DEC_SX32
#define COMET_DEC_SX32 4    // X ring depth for NT >= 32 (a shallower X ring leaves room for weights)
#endif
#ifndef COMET_DEC_WIDEN_WARPS
#define COMET_DEC_WIDEN_WARPS 8   // 8: two warps per TMEM lane quadrant (KS/2 K-blocks each); 4: one
#endif
#ifndef COMET_DEC_WIDEN_PF
#define COMET_DEC_WIDEN_PF 0   // 1: widen warps load stage s+1 weights before storing stage s (measured slower)
#endif
#ifndef COMET_DEC_EARLY_TRIGGER
#define COMET_DEC_EARLY_TRIGGER 0   // 1: trigger dependents at the start (measured slower)
#endif
#ifndef COMET_FIXUP_EARLY_TRIGGER
#define COMET_FIXUP_EARLY_TRIGGER 1
#endif
#ifndef COMET_DEC_SWMAX
#define COMET_DEC_SWMAX 8   // cap of the packed-weight ring depth (variant experiments)
#endif
#ifndef COMET_DEC_PDL
#define COMET_DEC_PDL 1     // launch as a programmatic dependent of kernel 1 (weights stream early)
#endif
constexpr int kWidenWarp0 = 4;
constexpr int kPromoWarp0 = 12;

// One pipeline stage = KS consecutive K-blocks of one tile (KS = 4 for NT <= 32, else 2), in
// two rings with their own barriers so the big weight slot is recycled as soon as it is read:
//   W ring  one box [8 row tiles][KS K-blocks][16 rows][64 B] of packed nibbles (64B swizzle);
//           released by the 8 widen warps right after their shared-memory loads.
//   X ring  one 3D box [KS K-blocks][NT tokens][128 B] of activation codes (SW128, the UMMA B
//           operand) + one 2D box [KS][NT] of per-token scales; released by the MMA commit and
//           the 4 promotion warps (which read the scales).
// Two producer threads (warp 0: W ring, warp 2: X ring).  Every widen warp takes part in every
// stage: warp 4 + 4h + q widens rows 32q .. 32q+31 of K-blocks [h KS/2, (h+1) KS/2).
// TMEM columns: [0, 2 * 32 KS) two widened-weight A buffers (alternate stages), then NACC
// accumulator sets of KS x NT columns (one accumulator per K-block of a stage).
template <int NT, bool GS = false, bool FQ = false>
struct Cfg {
  static constexpr int KS = NT <= 32 ? 4 : 2;                  // K-blocks per stage
  static constexpr int NA = COMET_DEC_NA;                       // widened-weight A buffers
  static constexpr int A_COLS = 32 * KS;
  static constexpr int ACC_SET = KS * NT;                      // accumulator columns per stage
  static constexpr int NACC_RAW = (512 - NA * A_COLS) / ACC_SET;
  static constexpr int NACC = NACC_RAW > 4 ? 4 : NACC_RAW;
  static constexpr uint32_t ACC_COL = NA * A_COLS;
  static constexpr int XKB_BYTES = NT * 128;                   // one K-block of codes
  static constexpr int W_BYTES = KS * kTileW * 64;             // KS K-blocks of packed weights
  static constexpr int S_BYTES = KS * NT * 4;
  // GS (group-wise weight scales): the X stage also carries the K-blocks' code sums qsum[b][m]
  // (int16, [KS][NT]) and weight scales s_w[b][n] (f32, [KS][128])
  // FQ (fused quantiser, comet_w4ax_linear): the in-kernel quantiser writes the codes, scales
  // and code sums of the stage here itself (the offset term is removed per block as in GS)
  static constexpr int Q_BYTES = (GS || FQ) ? KS * NT * 2 : 0;
  static constexpr int G_BYTES = GS ? KS * kTileW * 4 : 0;
  // FQ: the stage's raw 16-bit input rows (tokens < 8: the fused path serves M <= 8) land here
  // by TMA, [KS][8 rows][256 B]; the quantiser warp turns them into the codes above
  static constexpr int RAW_ROWS = 8;
  static constexpr int R_BYTES = FQ ? KS * RAW_ROWS * 256 : 0;
  static constexpr int X_STAGE = (KS * XKB_BYTES + S_BYTES + Q_BYTES + G_BYTES + R_BYTES + 1023) / 1024 * 1024;
  static constexpr int SX = NT >= 32 ? COMET_DEC_SX32 : 4;     // X ring depth
  static constexpr int SMEM_BUDGET = 224 * 1024;            // 227 KB minus alignment, barriers, tags
  static constexpr int SW_RAW = (SMEM_BUDGET - SX * X_STAGE) / W_BYTES;
  static constexpr int SW = SW_RAW > COMET_DEC_SWMAX ? COMET_DEC_SWMAX : SW_RAW;   // W ring depth
  static constexpr int SMEM_DATA = SW * W_BYTES + SX * X_STAGE;
  static constexpr int N_BARS = 2 * SW + 2 * SX + 2 * NA + 2 * NACC + (FQ ? SX : 0);
  static constexpr int SMEM_BYTES = 1024 + SMEM_DATA + N_BARS * 8 + 16 + kMaxBlocks;
  static constexpr int CH = NT < 32 ? NT : 32;                 // promotion column chunk
  static_assert(NT % 16 == 0 && NT <= 128, "decode tile");
  static_assert(NACC >= 1 && NACC * ACC_SET + NA * A_COLS <= 512, "TMEM budget");
  static_assert(SW >= 2 && SX >= 2, "ring depths");
  static_assert(SMEM_BYTES <= 227 * 1024, "shared memory budget");
};

template <int NCOL>
__device__ __forceinline__ void tmem_ld_cols(uint32_t taddr, uint32_t* r) {
  if constexpr (NCOL == 32) tmem_ld_32x32b_x32(taddr, r);
  else tmem_ld_32x32b_x16(taddr, r);
}

// GS (NEXT-3, reading R18): group-wise weight scales s_w[b][n], one per (128-channel block,
// output channel), given as w_scales [nb][N].  The weight scale no longer factors out of the K
// loop, so the promotion folds s_a[m,b] * s_w[b,n] per K-block and removes the offset-binary
// term per block: INT4 block  acc += s_a s_w (2^-9 sum q u - 2^-6 qsum)   (= s_a s_w 2^-9 sum q w)
//                 INT8 block  acc += s_a s_w 2^-13 (16 sum q w)
// and the epilogue only scales by 2^9.
template <int NT, int DEBUG, bool GS, bool FQ = false>
__global__ void __launch_bounds__(kThreads, 1) k_w4ax(const __grid_constant__ GemmParams P) {
  using C = Cfg<NT, GS, FQ>;
  constexpr int SW = C::SW;
  constexpr int SX = C::SX;
  constexpr int NA = C::NA;
  constexpr int NACC = C::NACC;
  constexpr int KS = C::KS;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // keep the pointer derived from the __shared__ array (shared address space) when aligning
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  auto sW = [&](int st) { return smem + st * C::W_BYTES; };
  auto sX = [&](int st) { return smem + SW * C::W_BYTES + st * C::X_STAGE; };
  auto sS = [&](int st) { return smem + SW * C::W_BYTES + st * C::X_STAGE + KS * C::XKB_BYTES; };
  auto sQ = [&](int st) { return sS(st) + C::S_BYTES; };          // GS only
  auto sG = [&](int st) { return sS(st) + C::S_BYTES + C::Q_BYTES; };
  auto sR = [&](int st) { return sS(st) + C::S_BYTES + C::Q_BYTES + C::G_BYTES; };   // FQ only
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + C::SMEM_DATA);
  uint64_t* full_w = bars;                  // [SW]   TMA -> widen
  uint64_t* empty_w = full_w + SW;          // [SW]   8 widen warps -> W producer
  uint64_t* full_x = empty_w + SW;          // [SX]   TMA -> (MMA, promotion)
  uint64_t* empty_x = full_x + SX;          // [SX]   MMA commit + 4 promotion warps -> X producer
  uint64_t* a_full = empty_x + SX;          // [NA]   8 widen warps -> MMA
  uint64_t* a_empty = a_full + NA;          // [NA]   MMA commit -> widen
  uint64_t* acc_full = a_empty + NA;        // [NACC] MMA commit -> promotion
  uint64_t* acc_empty = acc_full + NACC;    // [NACC] promotion -> MMA
  // FQ: full_x = the raw input landed (TMA -> quantiser), q_full = codes ready (quantiser ->
  // MMA and promotion); otherwise the consumers wait full_x (TMA of the codes) directly
  uint64_t* q_full = acc_empty + NACC;      // [SX] FQ only
  uint64_t* xready = FQ ? q_full : full_x;
  uint32_t* tmem_holder = reinterpret_cast<uint32_t*>(bars + C::N_BARS);
  uint8_t* s_tags = reinterpret_cast<uint8_t*>(tmem_holder + 4);
  const uint32_t s_tags_a = smem_u32(s_tags);
  // The CTA's work items, staged in shared memory at setup: every role walks the list, and a
  // global load of the next item at an item boundary costs microseconds once the weight stream
  // saturates HBM (it stalled the whole pipeline at every boundary).
  constexpr int kSmemItems = 64;
  __shared__ WorkItem s_items[kSmemItems];

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const bool debug = DEBUG != 0;
  const bool tracing = (COMET_DIAG || COMET_TRACE) && P.trace != nullptr;
  if (tracing && threadIdx.x == 0) P.trace[32768 + blockIdx.x * 4 + 0] = globaltimer_ns();
  const int it_begin = debug ? (int)blockIdx.x : P.cta_begin[blockIdx.x];
  const int it_end = debug ? (int)blockIdx.x + 1 : P.cta_begin[blockIdx.x + 1];
  const int nb = P.nb;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&P.map_x);
    tma_prefetch(&P.map_w);
    if (!FQ) tma_prefetch(&P.map_s);
    for (int i = 0; i < SW; ++i) {
      mbar_init(&full_w[i], 1);
      mbar_init(&empty_w[i], COMET_DEC_WIDEN_WARPS);
    }
    for (int i = 0; i < SX; ++i) {
      mbar_init(&full_x[i], 1);
      mbar_init(&empty_x[i], 1 + 4);
    }
    for (int i = 0; i < NA; ++i) {
      mbar_init(&a_full[i], COMET_DEC_WIDEN_WARPS);
      mbar_init(&a_empty[i], 1);
    }
    for (int i = 0; i < NACC; ++i) {
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_empty[i], 4);
    }
    if (FQ)
      for (int i = 0; i < SX; ++i) mbar_init(&q_full[i], 1);
    fence_mbar_init();
  }
  if (warp == 2) {
    tmem_alloc<512>(tmem_holder);
    tmem_relinquish();
  }
  for (int i = threadIdx.x; i < nb; i += kThreads) s_tags[i] = P.tags.get(i) ? 1 : 0;
  for (int i = threadIdx.x; i < min(kSmemItems, it_end - it_begin); i += kThreads) s_items[i] = load_item(P, it_begin + i, debug);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tbase = *tmem_holder;
  auto item = [&](int it) -> WorkItem {
    return it - it_begin < kSmemItems ? s_items[it - it_begin] : load_item(P, it, debug);
  };
  if (tracing && threadIdx.x == 0) P.trace[32768 + blockIdx.x * 4 + 1] = globaltimer_ns();
  int tr = 0;   // trace index (per role)
  // Programmatic dependent launch: the kernel may start while the previous kernel of the stream
  // (kernel 1, quantising this layer's activations) is still running.  Only the weight
  // producer -- it reads the packed weights and the plan, which no predecessor writes -- runs
  // ahead and fills the weight ring; every other thread first waits for the predecessor grid
  // to complete and its memory to be visible (a no-op without a programmatic predecessor).
  if (!(warp == 0 && lane == 0)) asm volatile("griddepcontrol.wait;" ::: "memory");
  // COMET_DEC_EARLY_TRIGGER: the next kernel of the stream (the fix-up kernel, or the next
  // layer's kernel) may launch now -- its CTAs take SMs as ours retire, so the tail of this grid
  // overlaps their start; they wait for our completion before touching our outputs
  if (COMET_DEC_EARLY_TRIGGER && threadIdx.x == 0) asm volatile("griddepcontrol.launch_dependents;");

  if (warp < kWidenWarp0) {
    setmaxnreg_dec<FQ ? 80 : 56>();
    if (warp == 0 && lane == 0) {
      // ------------------------------------------------------------------ W producer
      int st = 0;
      uint32_t ph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = item(it);
        const int n0 = (w.tile / P.n_m_tiles) * kTileW;
        for (int kb = w.kb_begin; kb < w.kb_end; kb += KS) {
          // one box per stage: KS K-blocks of the 128 rows, landing as [8 row tiles][KS][16][64 B]
          // (each row tile's KS K-blocks are contiguous in the packed layout: 8 requests of KS KB;
          // K-blocks past the tensor are zero-filled and counted)
          mbar_wait(&empty_w[st], ph ^ 1);
          mbar_arrive_expect_tx(&full_w[st], C::W_BYTES);
          tma_load_4d(sW(st), &P.map_w, &full_w[st], 0, 0, kb, n0 / kWTileRows);
          trace_ev(P, 0, tr++);
          if (++st == SW) { st = 0; ph ^= 1; }
        }
      }
    } else if (FQ && warp == 0 && lane == 1) {
      // ------------------------------------------------------------------ FQ raw-input producer
      int st = 0;
      uint32_t ph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = item(it);
        const int m0 = (w.tile % P.n_m_tiles) * NT;
        for (int kb = w.kb_begin; kb < w.kb_end; kb += KS) {
          mbar_wait(&empty_x[st], ph ^ 1);
          mbar_arrive_expect_tx(&full_x[st], C::R_BYTES);
          tma_load_3d(sR(st), &P.map_x, &full_x[st], 0, m0, kb);
          if (++st == SX) { st = 0; ph ^= 1; }
        }
      }
    } else if (FQ && (warp == 2 || warp == 3)) {
      // ------------------------------------------------------------------ fused quantiser (FQ)
      // Kernel 1 folded into the decode GEMM (comet_w4ax_linear, M <= 8): the stage's raw input
      // rows arrive by TMA (warp 0 lane 1, up to SX stages ahead); warps 2 and 3 take alternate
      // stages and quantise their (token, K-block) pairs from shared memory into the X slot, in the layout the codes' TMA would have
      // produced (codes [KS][NT][128 B] SW128, scales and code sums [KS][NT]), with kernel 1's
      // arithmetic (fmpq.cuh: identical codes, scales, code sums).  Four lanes per pair, 8 pairs
      // per round.  The offset-binary term is removed per block by the promotion (as for
      // group-wise scales): no per-row correction, every stream-K segment complete on its own.
      // Token rows >= M stay zero (the ring is zeroed first; a warp only ever touches its own
      // slots, j % SX with j of its parity, SX even).
      const int par = warp - 2;
      const int g = lane >> 2, sub = lane & 3;
      for (int i = par * 32 + lane; i < SX * C::X_STAGE / 16; i += 64)
        asm volatile("st.shared.v4.u32 [%0], {%1,%1,%1,%1};" ::"r"(smem_u32(sX(0)) + i * 16), "r"(0u) : "memory");
      __syncwarp();
      // stage cursor over the work list: (item, first K-block), global stage index j
      struct Cur { int it, kb, j; };
      auto advance = [&](Cur c) -> Cur {                  // the next stage
        const WorkItem w = item(c.it);
        c.kb += KS;
        ++c.j;
        if (c.kb >= w.kb_end) {
          ++c.it;
          if (c.it < it_end) c.kb = item(c.it).kb_begin;
        }
        return c;
      };
      Cur cur{it_begin, it_begin < it_end ? item(it_begin).kb_begin : 0, 0};
      if (par == 1 && cur.it < it_end) cur = advance(cur);
      while (cur.it < it_end) {
        Cur nxt = advance(cur);
        if (nxt.it < it_end) nxt = advance(nxt);          // this warp's next stage
        const WorkItem w = item(cur.it);
        const int st = cur.j % SX;
        const int64_t m0 = (int64_t)(w.tile % P.n_m_tiles) * NT;
        const int mrows = (int)min((int64_t)C::RAW_ROWS, P.M - m0);
        const int nk = min(KS, w.kb_end - cur.kb);
        mbar_wait(&full_x[st], (uint32_t)(cur.j / SX) & 1u);
        const int npairs = nk * mrows;
        for (int p0 = 0; p0 < npairs; p0 += 8) {
          const int pp = p0 + g;
          const bool pv = pp < npairs;
          const int kl = pv ? pp / mrows : 0, m = pv ? pp % mrows : 0;
          const uint32_t rsrc = smem_u32(sR(st)) + (kl * C::RAW_ROWS + m) * 256 + sub * 16;
          float v[32];
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const uint4 raw = lds128(rsrc + 64 * j);      // channels 32 j + 8 sub ..
            float t8[8];
            if (P.xq_bf16) fmpq::unpack8<true>(raw, t8); else fmpq::unpack8<false>(raw, t8);
#pragma unroll
            for (int i = 0; i < 8; ++i) v[8 * j + i] = t8[i];
          }
          const bool is8 = pv && lds_u8(s_tags_a + cur.kb + kl) != 0;
          const fmpq::LaneOut o = fmpq::quantize32(v, is8);   // every lane: quad shuffles
          if (pv) {
            const uint32_t rowb = smem_u32(sX(st)) + kl * C::XKB_BYTES + m * 128;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const int c0 = 32 * j + 8 * sub;              // byte of this lane's 8 codes in the row
              asm volatile("st.shared.v2.u32 [%0], {%1,%2};" ::"r"(rowb + ((((c0 >> 4) ^ (m & 7))) << 4) + (c0 & 15)),
                           "r"(o.c[j].x), "r"(o.c[j].y) : "memory");
            }
            if (sub == 0) {
              reinterpret_cast<float*>(sS(st))[kl * NT + m] = o.s;
              reinterpret_cast<int16_t*>(sQ(st))[kl * NT + m] = (int16_t)o.q;
            }
          }
        }
        fence_proxy_async_smem();                         // codes -> the MMA (async proxy)
        __syncwarp();
        if (lane == 0) mbar_arrive(&q_full[st]);
        cur = nxt;
      }
    } else if (!FQ && warp == 2 && lane == 0) {
      // ------------------------------------------------------------------ X producer
      int st = 0;
      uint32_t ph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = item(it);
        const int m0 = (w.tile % P.n_m_tiles) * NT;
        const int n0 = (w.tile / P.n_m_tiles) * kTileW;
        for (int kb = w.kb_begin; kb < w.kb_end; kb += KS) {
          mbar_wait(&empty_x[st], ph ^ 1);
          if (COMET_DEC_ABLATE & 16) {            // timing experiment: no activation loads
            mbar_arrive(&full_x[st]);
            if (++st == SX) { st = 0; ph ^= 1; }
            continue;
          }
          mbar_arrive_expect_tx(&full_x[st], KS * C::XKB_BYTES + C::S_BYTES + C::Q_BYTES + C::G_BYTES);
          tma_load_3d(sX(st), &P.map_x, &full_x[st], 0, m0, kb);
          tma_load_2d(sS(st), &P.map_s, &full_x[st], m0, kb);
          if (GS) {
            tma_load_2d(sQ(st), &P.map_q, &full_x[st], m0, kb);
            tma_load_2d(sG(st), &P.map_g, &full_x[st], n0, kb);
          }
          if (++st == SX) { st = 0; ph ^= 1; }
        }
      }
    } else if (warp == 1) {
      // ------------------------------------------------------------------ MMA issuer
      // The whole warp runs the loop and every operand is made warp-uniform (shuffle from lane
      // 0), so the compiler keeps the MMA operands in uniform registers; one elected lane
      // issues.  (With a lane-0-only loop every tcgen05.mma went through an R2UR waterfall.)
      // One K-block = 4 x tcgen05.mma (K = 32) into its own accumulator of the stage's set.
      const uint32_t id_f8 = idesc_f8f6f4_e4m3(128, NT);
      const uint32_t id_i8 = idesc_i8(128, NT);
      const uint32_t tb = __shfl_sync(0xffffffffu, tbase, 0);
      const uint32_t sx0 = __shfl_sync(0xffffffffu, smem_u32(sX(0)), 0);
      int sx = 0, ab = 0, accs = 0;
      uint32_t xph = 0, aph = 0, accph = 0;
      for (int it = it_begin; it < it_end; ++it) {
        const WorkItem w = item(it);
        const int kb_begin = __shfl_sync(0xffffffffu, w.kb_begin, 0);
        const int kb_end = __shfl_sync(0xffffffffu, w.kb_end, 0);
        for (int kb = kb_begin; kb < kb_end; kb += KS) {
          const int nk = min(KS, kb_end - kb);
          DEC_WAIT(2, &xready[sx], xph);
          DEC_WAIT(2, &a_full[ab], aph);
          DEC_WAIT(2, &acc_empty[accs], accph ^ 1);
          if (lane == 0) trace_ev(P, 1, tr);
          tc_fence_after();
          const uint32_t d0 = tb + C::ACC_COL + accs * C::ACC_SET;
          const uint32_t a0 = tb + ab * C::A_COLS;
          const uint64_t b0 = sdesc_kmajor_sw128(sx0 + sx * C::X_STAGE);
          const uint32_t tg = lane < KS ? lds_u8(s_tags_a + kb + lane) : 0u;
          const uint32_t tagw = __ballot_sync(0xffffffffu, tg != 0);
          // one elected thread issues the stage's MMAs AND its commits (tcgen05.commit tracks the
          // issuing thread's MMAs only)
          if (elect_one()) {
            for (int c = 0; c < nk; ++c) {
              const uint32_t d = d0 + c * NT, a = a0 + c * 32;
              const uint64_t bd = b0 + (uint64_t)((c * C::XKB_BYTES) >> 4);
              if (COMET_DEC_ABLATE & 1) {
              } else if ((tagw >> c) & 1u) {
#pragma unroll
                for (int k = 0; k < 4; ++k) mma_i8_ts(d, a + 8 * k, bd + 2 * k, id_i8, k);
              } else {
#pragma unroll
                for (int k = 0; k < 4; ++k) mma_f8_ts(d, a + 8 * k, bd + 2 * k, id_f8, k);
              }
            }
            tc_commit(&acc_full[accs]);
            tc_commit(&empty_x[sx]);
            tc_commit(&a_empty[ab]);
          }
          __syncwarp();
          if (lane == 0) trace_ev(P, 2, tr++);
          if (++sx == SX) { sx = 0; xph ^= 1; }
          if (++ab == NA) { ab = 0; aph ^= 1; }
          if (++accs == NACC) { accs = 0; accph ^= 1; }
        }
      }
    }
  } else if (warp < kPromoWarp0 && warp - kWidenWarp0 >= COMET_DEC_WIDEN_WARPS) {
    setmaxnreg_dec<112>();                        // spare warps of a 4-warp widen variant
  } else if (warp < kPromoWarp0) {
    setmaxnreg_dec<112>();
    // -------------------------------------------------------------------- widen (W -> TMEM A)
    constexpr int KH = KS * 4 / COMET_DEC_WIDEN_WARPS;   // K-blocks per widen warp and stage
    const int half = (warp - kWidenWarp0) >> 2;   // K-blocks [half KH, (half+1) KH) of a stage
    const int q = warp & 3;
    const int r = q * 32 + lane;                  // TMEM lane = weight row within the tile
    const uint32_t lane_addr = (uint32_t)(q * 32) << 16;
    // a stage's box lands as [8 row tiles][KS K-blocks][16 rows][64 B] (the packed layout's 1 KB
    // tiles, include/comet.h) with the TMA 64-byte swizzle: chunk ^= (row >> 1) & 3
    const int sw = (r >> 1) & 3;
    const uint32_t roff = (uint32_t)((r >> 4) * KS * 1024 + (r & 15) * 64);   // + cb KB
    int st = 0, ab = 0;
    uint32_t ph = 0, aph = 0;
    int seq = 0;
#if COMET_DEC_WIDEN_PF
    // Software-pipelined: the shared-memory loads of stage s+1's packed weights are issued
    // before stage s is converted and stored into TMEM, so their latency (~1000 clk when they
    // queue behind the previous stage's tcgen05.st in the memory pipe) overlaps the stores
    // instead of preceding them.
    int it = it_begin;
    WorkItem w{};
    int kb = 0;
    if (it < it_end) { w = item(it); kb = w.kb_begin; }
    uint4 cn[4 * KH];
    int kb_n = 0, nk_n = 0, seq_f = 0;
    auto fetch = [&]() {
      nk_n = min(KS, w.kb_end - kb);
      kb_n = kb;
      DEC_WAIT(4, &full_w[st], ph);
      if (lane == 0 && q == 0) trace_ev(P, 3 + half, seq_f);
#pragma unroll
      for (int i = 0; i < KH; ++i) {
        const int cb = half * KH + i;
        const uint32_t row = smem_u32(sW(st)) + roff + cb * 1024;
#pragma unroll
        for (int j = 0; j < 4; ++j)
          cn[4 * i + j] = (cb < nk_n && !(COMET_DEC_ABLATE & 8)) ? lds128(row + ((j ^ sw) << 4))
                                                                 : make_uint4(r, j, i, 0);
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty_w[st]);
      if (++st == SW) { st = 0; ph ^= 1; }
      ++seq_f;
      kb += KS;                                   // advance to the next stage of the work list
      if (kb >= w.kb_end) {
        ++it;
        if (it < it_end) { w = item(it); kb = w.kb_begin; }
      }
    };
    bool have = it < it_end;
    if (have) fetch();
    while (have) {
      uint4 cc[4 * KH];
#pragma unroll
      for (int i = 0; i < 4 * KH; ++i) cc[i] = cn[i];
      const int nk = nk_n, kbc = kb_n;
      const bool have_next = it < it_end;
      if (have_next) fetch();
      DEC_WAIT(4, &a_empty[ab], aph ^ 1);
      if (lane == 0 && q == 0 && half == 0) trace_ev(P, 14, seq);
      tc_fence_after();
#pragma unroll
      for (int i = 0; i < KH; ++i) {
        const int cb = half * KH + i;
        if (cb < nk) {
          const bool is8 = lds_u8(s_tags_a + kbc + cb) != 0;
          uint32_t o[32];
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const uint32_t pw[4] = {cc[4 * i + j].x, cc[4 * i + j].y, cc[4 * i + j].z, cc[4 * i + j].w};
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const uint32_t pv = pw[e];
              const int g = 2 * (j * 4 + e);
              widen_int4(pv, o[g], o[g + 1]);
              if (is8) {
                o[g] = int4_to_int8(o[g]);
                o[g + 1] = int4_to_int8(o[g + 1]);
              }
            }
          }
          if (!(COMET_DEC_ABLATE & 2)) tmem_st32(tbase + ab * C::A_COLS + cb * 32 + lane_addr, o);
        }
      }
      if (lane == 0 && q == 0 && half == 0) trace_ev(P, 13, seq);   // stores issued
      if (!(COMET_DEC_ABLATE & 2)) tmem_wait_st();
      if (lane == 0 && q == 0 && half == 0) trace_ev(P, 15, seq);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&a_full[ab]);
      if (lane == 0 && q == 0) trace_ev(P, 5 + half, seq);
      if (++ab == NA) { ab = 0; aph ^= 1; }
      ++seq;
      have = have_next;
    }
#else
    for (int it = it_begin; it < it_end; ++it) {
      const WorkItem w = item(it);
      for (int kb = w.kb_begin; kb < w.kb_end; kb += KS, ++seq) {
        const int nk = min(KS, w.kb_end - kb);
        DEC_WAIT(4, &full_w[st], ph);
        if (lane == 0 && q == 0) trace_ev(P, 3 + half, seq);
        // this warp's K-blocks of the stage: 4 x 16 B per K-block (row r, 128B-swizzled chunks)
        uint4 cc[4 * KH];
#pragma unroll
        for (int i = 0; i < KH; ++i) {
          const int cb = half * KH + i;
          const uint32_t row = smem_u32(sW(st)) + roff + cb * 1024;
#pragma unroll
          for (int j = 0; j < 4; ++j)
            cc[4 * i + j] = (cb < nk && !(COMET_DEC_ABLATE & 8)) ? lds128(row + ((j ^ sw) << 4))
                                                                 : make_uint4(r, j, i, 0);   // 8: diagnostic, no weight reads
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty_w[st]);
        DEC_WAIT(4, &a_empty[ab], aph ^ 1);
        if (lane == 0 && q == 0 && half == 0) trace_ev(P, 14, seq);
        tc_fence_after();
#if COMET_DEC_ST64
        if (KH == 2 && half * KH + 1 < nk) {
          // both K-blocks of this warp in one 64-column TMEM store
          uint32_t o[64];
#pragma unroll
          for (int i = 0; i < 2; ++i) {
            const bool is8 = lds_u8(s_tags_a + kb + half * KH + i) != 0;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const uint32_t pw[4] = {cc[4 * i + j].x, cc[4 * i + j].y, cc[4 * i + j].z, cc[4 * i + j].w};
#pragma unroll
              for (int e = 0; e < 4; ++e) {
                const uint32_t pv = pw[e];
                const int g = 32 * i + 2 * (j * 4 + e);
                widen_int4(pv, o[g], o[g + 1]);
                if (is8) {
                  o[g] = int4_to_int8(o[g]);
                  o[g + 1] = int4_to_int8(o[g + 1]);
                }
              }
            }
          }
          if (!(COMET_DEC_ABLATE & 2)) tmem_st64(tbase + ab * C::A_COLS + half * KH * 32 + lane_addr, o);
        } else
#endif
#pragma unroll
        for (int i = 0; i < KH; ++i) {
          const int cb = half * KH + i;
          if (cb < nk) {
            const bool is8 = lds_u8(s_tags_a + kb + cb) != 0;
            const uint32_t ta = tbase + ab * C::A_COLS + cb * 32 + lane_addr;
            uint32_t o[32];
            if (is8) {                          // warp-uniform, one branch per K-block
              widen_kblock_row<true>(&cc[4 * i], o);
              if (!(COMET_DEC_ABLATE & 2)) tmem_st32(ta, o);
            } else {
              widen_kblock_row<false>(&cc[4 * i], o);
              if (!(COMET_DEC_ABLATE & 2)) tmem_st32(ta, o);
            }
          }
        }
        if (lane == 0 && q == 0 && half == 0) trace_ev(P, 13, seq);   // stores issued
        if (!(COMET_DEC_ABLATE & 2)) tmem_wait_st();
        if (lane == 0 && q == 0 && half == 0) trace_ev(P, 15, seq);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&a_full[ab]);
        if (lane == 0 && q == 0) trace_ev(P, 5 + half, seq);
        if (++st == SW) { st = 0; ph ^= 1; }
        if (++ab == NA) { ab = 0; aph ^= 1; }
      }
    }
#endif
  } else {
    setmaxnreg_inc<208>();
    // -------------------------------------------------------------------- promotion + epilogue
    // TMEM accumulator: lane = weight row (n), column = token (m); 32x32b loads give thread t of
    // warp quarter q the row 32q + t and every token column of the tile.
    constexpr int CH = C::CH;
    const int q = warp & 3;
    const int row = q * 32 + lane;
    const uint32_t lane_addr = (uint32_t)(q * 32) << 16;
    const int ptid = threadIdx.x - kPromoWarp0 * 32;
    int sx = 0, accs = 0;
    uint32_t xph = 0, accph = 0;
    // Epilogue operands (s_w[n]; corr[m], the offset-binary correction of the owner segment) are
    // loaded ONE ITEM AHEAD into registers and first used at the next item: a global load
    // consumed at the start of an item stalls these warps for the load's latency -- microseconds
    // once the weight stream saturates HBM -- and with them the MMA and the whole stream.
    constexpr bool kEarlyCorr = NT <= 32 && !GS && !FQ; // registers: NT > 32 loads corr at the end
    float sw_nx = 0.f, cr_nx[kEarlyCorr ? NT : 1];
    auto prefetch_epi = [&](int it2) {
      if (it2 >= it_end) return;
      const WorkItem w2 = item(it2);
      const int64_t n2 = (int64_t)(w2.tile / P.n_m_tiles) * kTileW + row;
      const int64_t m2 = (int64_t)(w2.tile % P.n_m_tiles) * NT;
      if (!GS) sw_nx = ldg_nc_f32(P.w_scales + min(n2, P.N - 1));
      if constexpr (kEarlyCorr) {
#pragma unroll
        for (int j = 0; j < NT; ++j) cr_nx[j] = ldg_nc_f32(P.corr + min(m2 + j, P.Mp - 1));
      }
    };
    prefetch_epi(it_begin);
    for (int it = it_begin; it < it_end; ++it) {
      const WorkItem w = item(it);
      const int n_tile = w.tile / P.n_m_tiles, m_tile = w.tile % P.n_m_tiles;
      const int m0 = m_tile * NT, n0 = n_tile * kTileW;
      const bool owner = (w.flags & 2) != 0;
      const bool split = (w.flags & 1) != 0;
      const int n = n0 + row;
      const float sw_raw = sw_nx;
      float cr[kEarlyCorr ? NT : 1];
#pragma unroll
      for (int j = 0; j < (kEarlyCorr ? NT : 1); ++j) cr[j] = cr_nx[j];
      prefetch_epi(it + 1);
      float acc[NT];
      int32_t dacc[DEBUG ? NT : 1];
#pragma unroll
      for (int j = 0; j < NT; ++j) {
        acc[j] = 0.f;
        if (DEBUG) dacc[j] = 0;
      }
      for (int kb0 = w.kb_begin; kb0 < w.kb_end; kb0 += KS) {
        const int nk = min(KS, w.kb_end - kb0);
        DEC_WAIT(1, &xready[sx], xph);
        DEC_WAIT(1, &acc_full[accs], accph);
        if (ptid == 0) trace_ev(P, 7, tr);
        tc_fence_after();
        const uint32_t sbase = smem_u32(sS(sx));
        for (int c = 0; c < nk; ++c) {
          const int kb = kb0 + c;
          const bool is8 = lds_u8(s_tags_a + kb) != 0;
          float swb = 1.f;
          if (GS) asm volatile("ld.shared.f32 %0, [%1];" : "=f"(swb) : "r"(smem_u32(sG(sx)) + 4u * (c * kTileW + row)));
          const uint32_t tcol = tbase + C::ACC_COL + accs * C::ACC_SET + c * NT + lane_addr;
#pragma unroll
          for (int ch = 0; ch < NT / CH; ++ch) {
            uint32_t v[CH];
            if (COMET_DEC_ABLATE & 4) {
#pragma unroll
              for (int z = 0; z < CH; ++z) v[z] = 0;
            } else {
              tmem_ld_cols<CH>(tcol + ch * CH, v);
            }
            float sc[CH];
#pragma unroll
            for (int j = 0; j < CH; j += 4) {
              const float4 f = lds128f(sbase + (c * NT + ch * CH + j) * 4);
              sc[j] = f.x; sc[j + 1] = f.y; sc[j + 2] = f.z; sc[j + 3] = f.w;
            }
            if (GS) {
              // fold the block's weight scale into the per-token scales
#pragma unroll
              for (int j = 0; j < CH; ++j) sc[j] *= swb;
            }
            float qc[(GS || FQ) ? CH : 1];            // INT4 offset term 2^-6 qsum[b][m] (GS, FQ)
            if ((GS || FQ) && !is8) {
              // code sums of this K-block's tokens from the X stage (broadcast shared loads; the
              // box covers rows >= Mp with zeros)
              const uint32_t qa = smem_u32(sQ(sx)) + 2u * (c * NT + ch * CH);
#pragma unroll
              for (int j = 0; j < CH; j += 8) {
                const uint4 q8 = lds128(qa + 2u * j);
                const uint32_t qw[4] = {q8.x, q8.y, q8.z, q8.w};
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                  qc[j + 2 * e] = (float)(int16_t)(qw[e] & 0xFFFFu) * 0.015625f;
                  qc[j + 2 * e + 1] = (float)(int16_t)(qw[e] >> 16) * 0.015625f;
                }
              }
            }
            tmem_wait_ld();
            if (!is8) {
#pragma unroll
              for (int j = 0; j < CH; j += 2) {
                const int a = ch * CH + j;
                float2 vv = make_float2(__uint_as_float(v[j]), __uint_as_float(v[j + 1]));
                if (GS || FQ) vv = make_float2(vv.x - qc[j], vv.y - qc[j + 1]);   // exact: multiples of 2^-9 below 2^14
                const float2 y = ffma2(vv, make_float2(sc[j], sc[j + 1]), make_float2(acc[a], acc[a + 1]));
                acc[a] = y.x;
                acc[a + 1] = y.y;
              }
            } else {
#pragma unroll
              for (int j = 0; j < CH; j += 2) {
                const int a = ch * CH + j;
                const float2 s8 = make_float2(sc[j] * 1.220703125e-04f, sc[j + 1] * 1.220703125e-04f);  // 2^-13
                const float2 y = ffma2(i2f2_exact(v[j], v[j + 1]), s8, make_float2(acc[a], acc[a + 1]));
                acc[a] = y.x;
                acc[a + 1] = y.y;
              }
            }
            if (DEBUG) {
#pragma unroll
              for (int j = 0; j < CH; ++j) {
                const int64_t m = m0 + ch * CH + j;
                int32_t ab;
                if (is8) {
                  ab = ((int32_t)v[j]) >> 4;
                } else {
                  const int qs = (m < P.Mp) ? (int)P.qsum[(int64_t)kb * P.Mp + m] : 0;
                  ab = (int32_t)(__uint_as_float(v[j]) * 512.f) - 8 * qs;
                }
                dacc[ch * CH + j] += ab;
                if (DEBUG == 2 && m < P.M && n < P.N) P.dbg_blocks[((int64_t)kb * P.M + m) * P.N + n] = ab;
              }
            }
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&acc_empty[accs]);
          mbar_arrive(&empty_x[sx]);
        }
        if (ptid == 0) trace_ev(P, 8, tr++);
        if (++sx == SX) { sx = 0; xph ^= 1; }
        if (++accs == NACC) { accs = 0; accph ^= 1; }
      }
      // ---------------------------------------------------------------- epilogue
      if (ptid == 0) trace_ev(P, 10, it - it_begin);
      // the offset-binary correction -corr * 2^-9 belongs to the tile once: the owner segment
      // (K-block 0) folds it into its own sum
      const float swv = GS ? 512.f : (n < P.N ? sw_raw * 512.f : 0.f);
      if (!GS && !FQ && owner) {
#pragma unroll
        for (int j = 0; j < NT; ++j) {
          if constexpr (kEarlyCorr) acc[j] -= (m0 + j < P.Mp) ? cr[j] * 0.001953125f : 0.f;   // 2^-9
          else acc[j] -= (m0 + j < P.Mp) ? __ldg(P.corr + m0 + j) * 0.001953125f : 0.f;
        }
      }
      if (split) {
        // Stream-K fix-up off the pipeline: every segment of a split tile stores its
        // partial, already scaled by s_w (the owner's with the offset correction folded in),
        // into slot [fix][seg] -- only the tile's real token columns -- and moves on.  No fence,
        // atomic or wait: under a saturated HBM stream each gpu-scope round trip costs
        // microseconds and stalled this CTA's whole pipeline (tools/trace_dec.py).  The slots
        // are summed in segment order (deterministic) by k_fixup, a programmatic dependent launch
        // that starts when this grid has completed.
        const int seg = (w.flags >> 8) & 0xFF;
        const int64_t part4 = (int64_t)NT * kTileW / 4;
        const int nq = (int)((min((int64_t)NT, P.M - m0) + 3) / 4);   // float4 token groups stored
        float4* slot = reinterpret_cast<float4*>(P.ws_part) + ((int64_t)w.fix * P.max_seg + seg) * part4 + ptid;
#pragma unroll
        for (int j = 0; j < NT; j += 4)
          if (j / 4 < nq) slot[(j / 4) * 128] = make_float4(acc[j] * swv, acc[j + 1] * swv, acc[j + 2] * swv, acc[j + 3] * swv);
        if (ptid == 0) trace_ev(P, 12, it - it_begin);
        continue;
      }
      if (n < P.N) {
#pragma unroll
        for (int j = 0; j < NT; ++j) {
          const int64_t m = m0 + j;
          if (m < P.M) {
            const float yv = acc[j] * swv;
            const int64_t off = m * P.ldy + n;
            if (P.ydt == COMET_F16) reinterpret_cast<__half*>(P.y)[off] = __float2half_rn(yv);
            else if (P.ydt == COMET_BF16) reinterpret_cast<__nv_bfloat16*>(P.y)[off] = __float2bfloat16_rn(yv);
            else reinterpret_cast<float*>(P.y)[off] = yv;
            if (DEBUG) P.dbg_acc[m * P.N + n] = dacc[j];
          }
        }
      }
      if (ptid == 0) trace_ev(P, 12, it - it_begin);
    }
  }

  tc_fence_before();
  __syncthreads();
  // the fix-up kernel (programmatic dependent) may launch once every CTA got here; its
  // griddepcontrol.wait still waits for this grid's completion and memory flush
  if (!COMET_DEC_EARLY_TRIGGER) asm volatile("griddepcontrol.launch_dependents;");
  if (tracing && threadIdx.x == 0) {
    P.trace[32768 + blockIdx.x * 4 + 2] = globaltimer_ns();
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    P.trace[32768 + blockIdx.x * 4 + 3] = smid;
  }
  if (warp == 2) tmem_dealloc<512>(tbase);
}

// Stream-K fix-up of the decode kernel's split tiles: one CTA per split tile, thread = weight
// row; y[m, n] = sum over the tile's segments (in segment order) of the s_w-scaled partials.
template <int NT>
__global__ void __launch_bounds__(128) k_fixup(const __grid_constant__ GemmParams P, const int2* __restrict__ fix_info) {
  // let the next kernel of the stream (typically the next layer's GEMM, a programmatic
  // dependent) launch at once: its weight producer streams while this grid and the tail of the
  // GEMM before it run; its other threads wait for our completion
  if (COMET_FIXUP_EARLY_TRIGGER) asm volatile("griddepcontrol.launch_dependents;");
  asm volatile("griddepcontrol.wait;" ::: "memory");
  const int2 fi = fix_info[blockIdx.x];                 // {tile, segments}
  const int m0 = (fi.x % P.n_m_tiles) * NT, n0 = (fi.x / P.n_m_tiles) * kTileW;
  const int64_t n = n0 + threadIdx.x;
  const int64_t part4 = (int64_t)NT * kTileW / 4;
  const int nq = (int)((min((int64_t)NT, P.M - m0) + 3) / 4);
  const float4* slots = reinterpret_cast<const float4*>(P.ws_part) + (int64_t)blockIdx.x * P.max_seg * part4 + threadIdx.x;
  float4 acc[NT / 4];
#pragma unroll
  for (int j = 0; j < NT / 4; ++j) acc[j] = make_float4(0.f, 0.f, 0.f, 0.f);
  // slots in groups of G: all loads of a group in flight before the in-order adds (one slot
  // at a time made every slot a memory round trip: M = 32 decode GEMMs 40 -> 33 us)
  constexpr int G = NT <= 16 ? 8 : (NT <= 32 ? 4 : 2);
  for (int sg0 = 0; sg0 < fi.y; sg0 += G) {
    float4 t[G][NT / 4];
#pragma unroll
    for (int g = 0; g < G; ++g)
#pragma unroll
      for (int j = 0; j < NT / 4; ++j)
        t[g][j] = (sg0 + g < fi.y && j < nq) ? __ldcg(slots + (sg0 + g) * part4 + j * 128) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int g = 0; g < G; ++g)
#pragma unroll
      for (int j = 0; j < NT / 4; ++j) {
        if (sg0 + g >= fi.y) continue;
        acc[j].x += t[g][j].x; acc[j].y += t[g][j].y; acc[j].z += t[g][j].z; acc[j].w += t[g][j].w;
      }
  }
  if (n >= P.N) return;
#pragma unroll
  for (int j = 0; j < NT / 4; ++j) {
    const float v[4] = {acc[j].x, acc[j].y, acc[j].z, acc[j].w};
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      const int64_t m = m0 + 4 * j + t;
      if (j >= nq || m >= P.M) continue;
      const int64_t off = m * P.ldy + n;
      if (P.ydt == COMET_F16) reinterpret_cast<__half*>(P.y)[off] = __float2half_rn(v[t]);
      else if (P.ydt == COMET_BF16) reinterpret_cast<__nv_bfloat16*>(P.y)[off] = __float2bfloat16_rn(v[t]);
      else reinterpret_cast<float*>(P.y)[off] = v[t];
    }
  }
}

template <int NT>
cudaError_t launch_fixup(const GemmParams& prm, const int2* fix_info, int n_fix, cudaStream_t stream) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)n_fix);
  cfg.blockDim = dim3(128);
  cfg.dynamicSmemBytes = 0;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k_fixup<NT>, prm, fix_info);
}

template <int NT, int DEBUG, bool GS = false, bool FQ = false>
cudaError_t launch_nt(const GemmParams& prm, int grid, cudaStream_t stream) {
  using C = Cfg<NT, GS, FQ>;
  static std::atomic<uint64_t> attr_done{0};
  cudaError_t ea = set_smem_attr(k_w4ax<NT, DEBUG, GS, FQ>, C::SMEM_BYTES, attr_done);
  if (ea != cudaSuccess) return ea;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = C::SMEM_BYTES;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = COMET_DEC_PDL;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k_w4ax<NT, DEBUG, GS, FQ>, prm);
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
bool make_map(CUtensorMap* map, CUtensorMapDataType dt, int rank, const void* base,
              const uint64_t* dims, const uint64_t* stride_bytes, const uint32_t* box,
              CUtensorMapSwizzle swz) {
  auto fn = encode_fn();
  if (!fn) return false;
  cuuint64_t d[5], st[4];
  cuuint32_t bx[5], es[5];
  for (int i = 0; i < rank; ++i) { d[i] = dims[i]; bx[i] = box[i]; es[i] = 1; }
  for (int i = 0; i + 1 < rank; ++i) st[i] = stride_bytes[i];
  CUresult r = fn(map, dt, (cuuint32_t)rank, const_cast<void*>(base), d, st, bx, es,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

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

uint32_t next_epoch() {
  static std::atomic<uint32_t> g_epoch{0};
  uint32_t e = g_epoch.fetch_add(1, std::memory_order_relaxed) + 1;
  while (e == 0) e = g_epoch.fetch_add(1, std::memory_order_relaxed) + 1;   // 0 = zeroed flag
  return e;
}

// Diagnostic: the GEMM kernels' widening (widen_int4 / int4_to_int8) applied to the words
// first, first + 1, ... (mod 2^32); out[i] = {lo, hi} bytes of word first + i.
__global__ void k_debug_widen(uint64_t first, int64_t n, int is8, uint2* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    uint32_t lo, hi;
    widen_int4((uint32_t)(first + (uint64_t)i), lo, hi);
    if (is8) {
      lo = int4_to_int8(lo);
      hi = int4_to_int8(hi);
    }
    out[i] = make_uint2(lo, hi);
  }
}

cudaError_t launch_debug_widen(uint64_t first, int64_t n, int is8, uint32_t* out, cudaStream_t stream) {
  const int64_t blocks = std::min<int64_t>((n + 255) / 256, 148 * 16);
  k_debug_widen<<<(unsigned)std::max<int64_t>(blocks, 1), 256, 0, stream>>>(first, n, is8, reinterpret_cast<uint2*>(out));
  return cudaGetLastError();
}

}  // namespace gemm

// Persistent units of the plan's production kernel that can be co-resident on the current
// device: the stream-K fix-up waits of the persistent grid assume every unit is resident.
int max_coresident_units(const Plan& p, int sms) {
  using namespace gemm;
  if (p.orientation == 4) return p.num_ctas;   // no inter-CTA waits: any grid is valid
  if (p.orientation >= 2) return max_units_gemm_n(p.tile_w, p.orientation == 3 ? 2 : 1, sms);
  int b = 0;
  cudaError_t e = cudaSuccess;
  auto occ = [&](auto kern, int smem) {   // plan time: set the attribute directly (one lambda
                                          // instantiation serves every tile_n, so no cached flag)
    e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kern, kThreads, smem);
  };
  switch (p.tile_n) {
    case 16: occ(k_w4ax<16, 0, false>, Cfg<16>::SMEM_BYTES); break;
    case 32: occ(k_w4ax<32, 0, false>, Cfg<32>::SMEM_BYTES); break;
    case 64: occ(k_w4ax<64, 0, false>, Cfg<64>::SMEM_BYTES); break;
    default: occ(k_w4ax<128, 0, false>, Cfg<128>::SMEM_BYTES); break;
  }
  return e == cudaSuccess ? b * sms : -1;
}

// Shared-memory ring depth of the plan's production kernel (reported as plan_info.stages):
// prefill kernels: pipeline slots; decode kernel: packed-weight ring slots.
int gemm_stages(const Plan& p) {
  using namespace gemm;
  if (p.orientation == 4) return p.gemv_s;
  if (p.orientation >= 2) return stages_gemm_n(p.tile_w, p.orientation == 3 ? 2 : 1);
  switch (p.tile_n) {
    case 16: return Cfg<16>::SW;
    case 32: return Cfg<32>::SW;
    case 64: return Cfg<64>::SW;
    default: return Cfg<128>::SW;
  }
}

comet_status_t launch_gemm(Plan& p, const void* act_packed, const float* act_scales,
                           const void* w_packed, const float* w_scales, void* y,
                           comet_dtype_t ydt, int64_t ldy, int32_t* debug_acc,
                           int32_t* debug_acc_blocks, void* workspace, size_t ws_bytes,
                           cudaStream_t stream, int* launches, bool grouped, const RsArgs* rs,
                           const FusedX* fx) {
  using namespace gemm;
  if (fx && !(p.orientation == 4 || (p.orientation == 1 && p.tile_n == 16)) || (fx && (p.M > 8 || grouped || rs || debug_acc || debug_acc_blocks)))
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "the fused decode path needs M <= 8 and orientation 4, or orientation 1 with 16-token tiles");
  static_assert(Cfg<16, false, true>::SX % 2 == 0, "the fused quantiser's two warps own alternate X slots");
  if (grouped && p.orientation != 1 && !(p.orientation == 3 && p.tile_w == 256))
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "group-wise weight scales run on orientation 1 or on the 256-wide pair kernel (orientation 3)");
  if (grouped && p.orientation == 3 && (debug_acc || debug_acc_blocks))
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "group-wise weight scales on the pair kernel have no debug accumulators");
  *launches = 0;
  if (p.orientation == 4) {
    if (grouped || rs || debug_acc || debug_acc_blocks)
      return fail(COMET_ERR_UNSUPPORTED_SHAPE, "orientation 4 (decode, M <= 8) runs per-channel weight scales without debug outputs");
    if (p.d_items == nullptr) return fail(COMET_ERR_INVALID_ARG, "plan was created with device_plan = 0");
    if (workspace == nullptr || ws_bytes < p.ws_bytes)
      return fail(COMET_ERR_WORKSPACE_TOO_SMALL, "workspace smaller than the plan's workspace_bytes");
    comet_act_layout_t L;
    act_layout(p.M, p.K, &L);
    const uint8_t* base = static_cast<const uint8_t*>(act_packed);
    // fx (comet_w4ax_linear): the kernel quantises x itself -- one launch + the reduction
    cudaError_t e = gemv::launch_gemv(static_cast<const uint8_t*>(w_packed), fx ? nullptr : base + L.codes_off,
                                      act_scales, fx ? nullptr : reinterpret_cast<const int16_t*>(base + L.qsum_off),
                                      w_scales, y, (int)ydt, ldy, p.M, p.N, p.K, L.Mp, p.mask, p.num_ctas,
                                      p.max_segments, p.gemv_nbr, p.gemv_s, static_cast<float*>(workspace), stream,
                                      fx ? fx->x : nullptr, fx ? fx->ldx : 0, fx ? fx->bf16 : false);
    if (e != cudaSuccess) return cuda_status(e, "w4ax gemv launch");
    *launches = 2;
    return COMET_OK;
  }
  const bool dbg = debug_acc != nullptr || debug_acc_blocks != nullptr;
  const int debug = debug_acc_blocks ? 2 : (dbg ? 1 : 0);
  const bool normal = p.orientation >= 2;
  const int cg = p.orientation == 3 ? 2 : 1;
  // token-tile and weight-tile of one CTA (= box rows of the two TMA maps) and of the tile
  int tile_m, tile_w, cta_rows_w;
  if (normal) { tile_m = 128 * cg; tile_w = dbg ? 96 : p.tile_w; cta_rows_w = tile_w / cg; }
  else { tile_m = dbg ? 32 : p.tile_n; tile_w = kTileW; cta_rows_w = kTileW; }
  const int box_m = normal ? 128 : tile_m;
  comet_act_layout_t L;
  act_layout(p.M, p.K, &L);
  const uint8_t* base = static_cast<const uint8_t*>(act_packed);
  GemmParams prm;
  memset(&prm, 0, sizeof(prm));
  if (normal) {
    if (!make_map_2d(&prm.map_x, base + L.codes_off, (uint64_t)p.K, (uint64_t)p.M, (uint64_t)p.K, 128,
                     (uint32_t)box_m, CU_TENSOR_MAP_SWIZZLE_128B))
      return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the activation codes");
  } else if (fx) {
    // the raw input as [nb][M][128 halves] (dims innermost first: channel in block, token,
    // block), one box of [KS][8 tokens][256 B] per stage (rows >= M are zero-filled)
    const uint64_t rd[3] = {128, (uint64_t)p.M, (uint64_t)p.nb};
    const uint64_t rs_[2] = {(uint64_t)fx->ldx * 2, 256};
    const uint32_t rb[3] = {128, 8, (uint32_t)(tile_m <= 32 ? 4 : 2)};
    if (!make_map(&prm.map_x, CU_TENSOR_MAP_DATA_TYPE_UINT16, 3, fx->x, rd, rs_, rb, CU_TENSOR_MAP_SWIZZLE_NONE))
      return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the fused path's input");
    prm.xq = fx->x;
    prm.ldxq = fx->ldx;
    prm.xq_bf16 = fx->bf16 ? 1 : 0;
  } else {
    // decode: codes as [nb][M][128 B] (dims innermost first: byte in block, token, block) so
    // one box brings a stage's KS K-blocks as KS UMMA-ready [NT][128 B] SW128 tiles; scales
    // [nb][Mp] f32, one box of KS x NT per stage.
    const uint32_t ks = tile_m <= 32 ? 4 : 2;
    const uint64_t xd[3] = {128, (uint64_t)p.M, (uint64_t)p.nb};
    const uint64_t xs[2] = {(uint64_t)p.K, 128};
    const uint32_t xb[3] = {128, (uint32_t)tile_m, ks};
    if (!make_map(&prm.map_x, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, base + L.codes_off, xd, xs, xb,
                  CU_TENSOR_MAP_SWIZZLE_128B))
      return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the activation codes (3D)");
    const uint64_t sd[2] = {(uint64_t)L.Mp, (uint64_t)p.nb};
    const uint64_t ss[1] = {(uint64_t)L.Mp * 4};
    const uint32_t sb[2] = {(uint32_t)tile_m, ks};
    if (!make_map(&prm.map_s, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, act_scales, sd, ss, sb,
                  CU_TENSOR_MAP_SWIZZLE_NONE))
      return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the activation scales");
    if (grouped) {
      // qsum [nb][Mp] int16, box KS x NT; grouped weight scales [nb][N] f32, box KS x 128
      const uint64_t qs[1] = {(uint64_t)L.Mp * 2};
      if (!make_map(&prm.map_q, CU_TENSOR_MAP_DATA_TYPE_UINT16, 2, base + L.qsum_off, sd, qs, sb,
                    CU_TENSOR_MAP_SWIZZLE_NONE))
        return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the code sums");
      const uint64_t gd[2] = {(uint64_t)p.N, (uint64_t)p.nb};
      const uint64_t gs[1] = {(uint64_t)p.N * 4};
      const uint32_t gb[2] = {(uint32_t)kTileW, ks};
      if (!make_map(&prm.map_g, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, w_scales, gd, gs, gb,
                    CU_TENSOR_MAP_SWIZZLE_NONE))
        return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the group-wise weight scales");
    }
  }
  // packed weights as [N/16 row tiles][nb K-blocks][16 rows][64 B] (dims innermost first), 64B
  // swizzle; prefill: one K-block of the CTA's rows per box, decode: a stage's KS K-blocks of 128
  // rows (KS = 4 for tiles of <= 32 tokens, else 2)
  {
    const uint64_t wd[4] = {64, (uint64_t)kWTileRows, (uint64_t)p.nb, (uint64_t)(p.N / kWTileRows)};
    const uint64_t ws_[3] = {64, 64 * kWTileRows, (uint64_t)p.nb * 64 * kWTileRows};
    const uint32_t wb[4] = {64, (uint32_t)kWTileRows, normal ? 1u : (tile_m <= 32 ? 4u : 2u),
                            (uint32_t)(cta_rows_w / kWTileRows)};
    if (!make_map(&prm.map_w, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, w_packed, wd, ws_, wb, CU_TENSOR_MAP_SWIZZLE_64B))
      return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the packed weights");
  }
  if (normal && !dbg) {
    const int esz = ydt == COMET_F32 ? 4 : 2;
    if (!make_map_2d(&prm.map_y, y, (uint64_t)p.N * esz, (uint64_t)p.M, (uint64_t)ldy * esz, 64,
                     COMET_EPI_WARP ? 32 : 128,
                     CU_TENSOR_MAP_SWIZZLE_64B))
      return fail(COMET_ERR_CUDA, "cuTensorMapEncodeTiled failed for the output");
  }
  prm.scales = act_scales;
  prm.corr = fx ? nullptr : reinterpret_cast<const float*>(base + L.corr_off);
  prm.qsum = fx ? nullptr : reinterpret_cast<const int16_t*>(base + L.qsum_off);
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
  if (rs) {
    prm.rs_world = rs->world;
    prm.rs_rank = rs->rank;
    prm.rs_ms = rs->ms;
    for (int i = 0; i < 8; ++i) prm.rs_dst[i] = i < rs->world ? rs->dst[i] : nullptr;
  }
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
    prm.epoch = next_epoch();
    grid = p.num_ctas * cg;
  }
  if (normal) {
    e = launch_gemm_n(prm, grid, tile_w, cg, debug, stream, grouped);
  } else if (dbg) {
    if (grouped) e = debug == 2 ? launch_nt<32, 2, true>(prm, grid, stream) : launch_nt<32, 1, true>(prm, grid, stream);
    else e = debug == 2 ? launch_nt<32, 2>(prm, grid, stream) : launch_nt<32, 1>(prm, grid, stream);
  } else if (grouped) {
    switch (tile_m) {
      case 16: e = launch_nt<16, 0, true>(prm, grid, stream); break;
      case 32: e = launch_nt<32, 0, true>(prm, grid, stream); break;
      case 64: e = launch_nt<64, 0, true>(prm, grid, stream); break;
      case 128: e = launch_nt<128, 0, true>(prm, grid, stream); break;
      default: return fail(COMET_ERR_UNSUPPORTED_SHAPE, "unsupported tile_n");
    }
  } else if (fx) {
    e = launch_nt<16, 0, false, true>(prm, grid, stream);
  } else {
    switch (tile_m) {
      case 16: e = launch_nt<16, 0>(prm, grid, stream); break;
      case 32: e = launch_nt<32, 0>(prm, grid, stream); break;
      case 64: e = launch_nt<64, 0>(prm, grid, stream); break;
      case 128: e = launch_nt<128, 0>(prm, grid, stream); break;
      default: return fail(COMET_ERR_UNSUPPORTED_SHAPE, "unsupported tile_n");
    }
  }
  if (e != cudaSuccess) return cuda_status(e, "w4ax gemm launch");
  *launches = 1;
  if (!normal && !dbg && p.n_split_tiles > 0) {
    // the decode kernel's split tiles are summed by the fix-up kernel
    const int2* fi = reinterpret_cast<const int2*>(p.d_fix);
    const int nf = (int)p.n_split_tiles;
    switch (tile_m) {
      case 16: e = launch_fixup<16>(prm, fi, nf, stream); break;
      case 32: e = launch_fixup<32>(prm, fi, nf, stream); break;
      case 64: e = launch_fixup<64>(prm, fi, nf, stream); break;
      default: e = launch_fixup<128>(prm, fi, nf, stream); break;
    }
    if (e != cudaSuccess) return cuda_status(e, "fix-up launch");
    *launches = 2;
  }
  return COMET_OK;
}

// NEXT-2: the owner's side of the fused reduce-scatter -- y[m][n] = sum over source ranks, in rank
// order (deterministic), of recv[src][m][n]; FP32 in, F16 / BF16 / F32 out.  HBM-bound.
__global__ void __launch_bounds__(256) k_rs_reduce(const float4* __restrict__ recv, int world, int64_t rows,
                                                   int64_t ms, int64_t N, void* y, int ydt, int64_t ldy) {
  const int64_t n4 = N / 4, total = rows * n4, plane = ms * n4;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    float4 acc = __ldcs(recv + i);
    for (int s = 1; s < world; ++s) {
      const float4 t = __ldcs(recv + s * plane + i);
      acc.x += t.x; acc.y += t.y; acc.z += t.z; acc.w += t.w;
    }
    const int64_t m = i / n4, n = (i - m * n4) * 4;
    if (ydt == COMET_F32) {
      *reinterpret_cast<float4*>(reinterpret_cast<float*>(y) + m * ldy + n) = acc;
    } else if (ydt == COMET_BF16) {
      __nv_bfloat162 a = __floats2bfloat162_rn(acc.x, acc.y), b = __floats2bfloat162_rn(acc.z, acc.w);
      *reinterpret_cast<uint2*>(reinterpret_cast<__nv_bfloat16*>(y) + m * ldy + n) =
          make_uint2(*reinterpret_cast<uint32_t*>(&a), *reinterpret_cast<uint32_t*>(&b));
    } else {
      __half2 a = __floats2half2_rn(acc.x, acc.y), b = __floats2half2_rn(acc.z, acc.w);
      *reinterpret_cast<uint2*>(reinterpret_cast<__half*>(y) + m * ldy + n) =
          make_uint2(*reinterpret_cast<uint32_t*>(&a), *reinterpret_cast<uint32_t*>(&b));
    }
  }
}

cudaError_t launch_rs_reduce(const float* recv, int world, int64_t rows, int64_t ms, int64_t N, void* y, int ydt,
                             int64_t ldy, cudaStream_t stream) {
  const int64_t total = rows * (N / 4);
  if (total == 0) return cudaSuccess;
  const int64_t blocks = std::min<int64_t>((total + 255) / 256, 148 * 8);
  k_rs_reduce<<<(unsigned)blocks, 256, 0, stream>>>(reinterpret_cast<const float4*>(recv), world, rows, ms, N, y, ydt, ldy);
  return cudaGetLastError();
}

}  // namespace comet
