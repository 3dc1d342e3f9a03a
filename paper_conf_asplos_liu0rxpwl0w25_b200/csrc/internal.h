// internal.h -- declarations shared by the libcomet.so translation units (not part of the ABI).
#pragma once
#include <algorithm>
#include <cstdint>
#include <cstddef>
#include <string>
#include <vector>
#include <atomic>
#include <cuda_runtime.h>

#include "../../include/comet.h"

namespace comet {

constexpr int kBlockK = 128;       // FMPQ block
constexpr int kTileW = 128;        // weight rows per output tile = MMA M (one CTA, cta_group::1)
constexpr int kMaxBlocks = 1024;   // K <= 131072

// 1024-bit tag mask passed by value to kernels.
struct TagMask {
  uint32_t w[kMaxBlocks / 32];
  __host__ __device__ bool get(int b) const { return (w[b >> 5] >> (b & 31)) & 1u; }
};

// Packed weights are row-tiled (include/comet.h): 1 KB tiles of 16 rows x one K-block (64 B
// per row), tile (n/16, b) at ((n/16) * nb + b) KB.  Word g (channels 8g .. 8g+7) of row n:
__host__ __device__ inline int64_t packed_word_index(int64_t n, int64_t g, int64_t nb) {
  return ((((n >> 4) * nb + (g >> 4)) << 4) + (n & 15)) * 16 + (g & 15);
}
constexpr int kWTileRows = 16;     // rows per packed-weight tile

inline int64_t round_up(int64_t a, int64_t b) { return (a + b - 1) / b * b; }
inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Work item of the persistent GEMM: one output tile, a half-open K-block range.
// flags: bit0 = tile is split across CTAs, bit1 = this item owns the tile (holds kb 0, does
// the fix-up and the store); bits 8..15 = segment index within the tile (0 = owner);
// bits 16..23 = number of segments of the tile.  fix = index of the tile among split tiles.
struct WorkItem {
  int32_t tile, kb_begin, kb_end, flags;
  int32_t fix, pad0, pad1, pad2;
};
static_assert(sizeof(WorkItem) == 32, "work item layout");

struct Plan {
  int64_t M, N, K, nb, Mp;
  int tile_n, num_ctas, split_mode, stages;
  int orientation = 1;   // 1: weights on MMA M (gemm.cu), 2: tokens on MMA M (gemm_n.cu)
  int tile_w = 128;      // weights per output tile
  int kgran = 1;         // K-blocks per scheduling unit (4 for the decode kernel's stream-K)
  int gemv_nbr = 0;      // orientation 4: activation K-blocks one CTA stages
  int gemv_s = 0;        // orientation 4: weight ring depth (K-blocks in flight per warp)
  int64_t n_m_tiles, n_n_tiles, n_tiles;
  std::vector<uint8_t> tags;
  TagMask mask;
  std::vector<int32_t> cta_begin;       // [num_ctas + 1] offsets into items
  std::vector<WorkItem> items;
  int64_t n_split_tiles = 0;
  int max_segments = 1;
  double max_cost = 0, mean_cost = 0;
  // device copies
  int32_t* d_cta_begin = nullptr;
  WorkItem* d_items = nullptr;
  std::vector<int32_t> fix_info;        // [n_split_tiles][2] = {tile, segments} (fix order)
  int32_t* d_fix = nullptr;
  size_t ws_bytes = 0;                  // stream-K partials + flags
  size_t ws_flags_off = 0;
  int device = -1;
};

// thread-local error detail
void set_error(const std::string& msg);
comet_status_t fail(comet_status_t st, const std::string& msg);
comet_status_t cuda_status(cudaError_t e, const char* what);
void note_launches(int n);

// planner.cpp
comet_status_t build_plan(Plan& p, const comet_sched_config& cfg);

// quantize.cu
cudaError_t launch_quantize(const void* x, bool bf16, int64_t M, int64_t K, int64_t ldx,
                            const TagMask& tags, void* act_packed, float* act_scales,
                            cudaStream_t stream, int* launches);
cudaError_t launch_quantize_perm(const void* x, bool bf16, int64_t M, int64_t K, int64_t ldx,
                                 const TagMask& tags, const int32_t* perm, void* act_packed,
                                 float* act_scales, cudaStream_t stream, int* launches);
cudaError_t launch_pack_weight_perm(const int8_t* w, int64_t N, int64_t K, const int32_t* perm,
                                    void* w_packed, cudaStream_t stream);
cudaError_t launch_channel_amax(const void* x, bool bf16, int64_t M, int64_t K, int64_t ldx,
                                float* amax, cudaStream_t stream);
// kv4.cu (NEXT-4)
cudaError_t launch_kv4_quantize(const void* x, bool bf16, int64_t T, int64_t C, int64_t ldx, int G,
                                uint8_t* codes, float* scales, float* mins, cudaStream_t stream);
cudaError_t launch_kv4_dequantize(const uint8_t* codes, const float* scales, const float* mins,
                                  int64_t T, int64_t C, int G, void* y, bool bf16, int64_t ldy,
                                  cudaStream_t stream);
// pack.cu
cudaError_t launch_pack_weight(const int8_t* w, int64_t N, int64_t K, void* w_packed,
                               cudaStream_t stream);
// gemm.cu
// comet_w4ax_linear's fused decode path: the GEMM quantises x itself (no kernel 1)
struct FusedX {
  const void* x;
  int64_t ldx;
  bool bf16;
};

struct RsArgs {            // NEXT-2 fused reduce-scatter of the row-parallel layer
  int world, rank;
  int64_t ms;              // output rows per owner rank
  float* dst[8];           // every rank's receive buffer [world][ms][N] (peer-mapped pointers)
};
comet_status_t launch_gemm(Plan& p, const void* act_packed, const float* act_scales,
                           const void* w_packed, const float* w_scales, void* y,
                           comet_dtype_t ydt, int64_t ldy, int32_t* debug_acc,
                           int32_t* debug_acc_blocks, void* workspace, size_t ws_bytes,
                           cudaStream_t stream, int* launches, bool grouped = false,
                           const RsArgs* rs = nullptr, const FusedX* fx = nullptr);
cudaError_t launch_rs_reduce(const float* recv, int world, int64_t rows, int64_t ms, int64_t N, void* y, int ydt,
                             int64_t ldy, cudaStream_t stream);
int max_coresident_units(const Plan& p, int sms);
int gemm_stages(const Plan& p);
// gemm_v.cu: the decode-regime kernel of plan orientation 4 (M <= 8)
namespace gemv {
int gemv_ctas_per_sm();
int gemv_stages();
int gemv_max_segments(int64_t units, int nb, int ctas);
int gemv_stage_blocks(int64_t units, int nb, int ctas);
int gemv_pick(int64_t M, int64_t units, int nb, int num_sms, int* nbr_out, int* s_out);
cudaError_t launch_gemv(const uint8_t* w, const uint8_t* codes, const float* scales, const int16_t* qsum,
                        const float* w_scales, void* y, int ydt, int64_t ldy, int64_t M, int64_t N,
                        int64_t K, int64_t Mp, const TagMask& tags, int ctas, int maxseg, int nbr,
                        int S, float* part, cudaStream_t stream, const void* x = nullptr, int64_t ldx = 0,
                        bool xbf16 = false);
}
namespace gemm {
cudaError_t launch_debug_widen(uint64_t first, int64_t n, int is8, uint32_t* out, cudaStream_t stream);
}
// act layout
void act_layout(int64_t M, int64_t K, comet_act_layout_t* out);

}  // namespace comet
