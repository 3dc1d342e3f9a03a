// api.cu -- the C ABI of libcomet.so (include/comet.h): validation, layouts, planning, dispatch.
#include <cstring>
#include <cstdio>
#include <mutex>
#include <new>
#include "internal.h"
#include "gemm_common.cuh"

struct comet_plan_s {
  comet::Plan p;
  comet_sched_config cfg{};          // as resolved at create time (sub-plans reuse it)
  // comet_w4ax_linear_host pipeline: token chunks of kLinChunk rows, each with its own H2D copy,
  // quantise + GEMM and D2H copy on three streams, so the PCIe transfers of neighbouring chunks
  // overlap each other (full duplex) and the compute.  Created on first use.
  comet_plan_s* chunk = nullptr;     // sub-plan, M = kLinChunk
  comet_plan_s* tail = nullptr;      // sub-plan, M = M % kLinChunk (when nonzero)
  cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
  std::vector<cudaEvent_t> ev;       // [3 per chunk]: H2D done, compute done, D2H done; + 2:
                                     // last quantise of the previous call, its last D2H
  bool prev_call = false;            // the two events above were recorded
  void* ws_zeroed = nullptr;         // scratch address whose fix-up workspace was last zeroed
};

namespace comet {

static thread_local std::string g_err;
static thread_local int g_launches = 0;

void set_error(const std::string& msg) { g_err = msg; }
comet_status_t fail(comet_status_t st, const std::string& msg) {
  g_err = msg;
  return st;
}
comet_status_t cuda_status(cudaError_t e, const char* what) {
  g_err = std::string(what) + ": " + cudaGetErrorString(e);
  return COMET_ERR_CUDA;
}
void note_launches(int n) { g_launches = n; }

static comet_status_t check_device(int* sms = nullptr) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_status(e, "cudaGetDevice");
  int major = 0, minor = 0, nsm = 0;
  cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev);
  cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  if (major != 10 || minor != 0)
    return fail(COMET_ERR_NOT_SM100A, "libcomet.so needs an sm_100a (B200) device; found sm_" +
                                          std::to_string(major) + std::to_string(minor));
  if (sms) *sms = nsm;
  return COMET_OK;
}

static bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

static comet_status_t check_mk(int64_t M, int64_t K) {
  if (M < 1 || M > INT32_MAX) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "M must be in [1, 2^31-1]");
  if (K < kBlockK || K % kBlockK != 0 || K > (int64_t)kBlockK * kMaxBlocks)
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "K must be a positive multiple of 128, <= 131072");
  return COMET_OK;
}
static comet_status_t check_n(int64_t N) {
  if (N < kTileW || N % kTileW != 0 || N > (1 << 20))
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "N must be a positive multiple of 128, <= 2^20");
  return COMET_OK;
}

static TagMask mask_of(const uint8_t* tags, int64_t nb) {
  TagMask m;
  memset(&m, 0, sizeof(m));
  for (int64_t b = 0; b < nb; ++b)
    if (tags[b]) m.w[b >> 5] |= 1u << (b & 31);
  return m;
}

}  // namespace comet

using namespace comet;

extern "C" {

const char* comet_status_string(comet_status_t s) {
  switch (s) {
    case COMET_OK: return "COMET_OK";
    case COMET_ERR_INVALID_ARG: return "COMET_ERR_INVALID_ARG";
    case COMET_ERR_UNSUPPORTED_SHAPE: return "COMET_ERR_UNSUPPORTED_SHAPE";
    case COMET_ERR_MISALIGNED: return "COMET_ERR_MISALIGNED";
    case COMET_ERR_NOT_SM100A: return "COMET_ERR_NOT_SM100A";
    case COMET_ERR_WORKSPACE_TOO_SMALL: return "COMET_ERR_WORKSPACE_TOO_SMALL";
    case COMET_ERR_CUDA: return "COMET_ERR_CUDA";
  }
  return "COMET_ERR_UNKNOWN";
}

const char* comet_last_error(void) { return g_err.c_str(); }
const char* comet_version(void) { return "comet-b200 0.1 (sm_100a; W4Ax = FP8-exact INT4 blocks + INT8 blocks)"; }
int comet_last_launch_count(void) { return g_launches; }

/* Diagnostic (not part of comet.h): subsequent GEMM launches record a clock64 timeline of the
 * first two CTAs into buf ([2][8][1024] uint64, device memory); NULL disables. */
void comet_debug_set_trace(void* buf) { comet::gemm::g_trace = static_cast<unsigned long long*>(buf); }

comet_status_t comet_debug_widen(uint64_t first_word, int64_t n, int int8_block, uint32_t* out_dev,
                                 void* stream) {
  g_launches = 0;
  if (n < 0 || n > ((int64_t)1 << 32)) return fail(COMET_ERR_INVALID_ARG, "n must be in [0, 2^32]");
  if (n == 0) return COMET_OK;
  if (!out_dev) return fail(COMET_ERR_INVALID_ARG, "out_dev is NULL");
  if ((reinterpret_cast<uintptr_t>(out_dev) & 7u) != 0) return fail(COMET_ERR_MISALIGNED, "out_dev must be 8-byte aligned");
  comet_status_t st = check_device();
  if (st != COMET_OK) return st;
  cudaError_t e = gemm::launch_debug_widen(first_word, n, int8_block ? 1 : 0, out_dev, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_status(e, "widen launch");
  g_launches = 1;
  return COMET_OK;
}

comet_status_t comet_act_layout(int64_t M, int64_t K, comet_act_layout_t* out) {
  if (!out) return fail(COMET_ERR_INVALID_ARG, "out is NULL");
  comet_status_t st = check_mk(M, K);
  if (st != COMET_OK) return st;
  act_layout(M, K, out);
  return COMET_OK;
}

size_t comet_act_packed_bytes(int64_t M, int64_t K) {
  if (check_mk(M, K) != COMET_OK) return 0;
  comet_act_layout_t L;
  act_layout(M, K, &L);
  return L.total_bytes;
}

size_t comet_act_scales_count(int64_t M, int64_t K) {
  if (check_mk(M, K) != COMET_OK) return 0;
  return (size_t)(K / kBlockK) * (size_t)round_up(M, COMET_SCALE_PAD);
}

comet_status_t comet_quantize_act(const void* x, comet_dtype_t xdt, int64_t M, int64_t K,
                                  int64_t ldx, const uint8_t* tags_host, const int32_t* perm_dev,
                                  void* act_packed, float* act_scales, void* stream) {
  g_launches = 0;
  comet_status_t st = check_mk(M, K);
  if (st != COMET_OK) return st;
  if (!x || !tags_host || !act_packed || !act_scales) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (xdt != COMET_F16 && xdt != COMET_BF16) return fail(COMET_ERR_INVALID_ARG, "xdt must be COMET_F16 or COMET_BF16");
  if (perm_dev && K > 32768) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "the fused channel permutation needs K <= 32768");
  if (perm_dev && !aligned16(perm_dev)) return fail(COMET_ERR_MISALIGNED, "perm_dev must be 16-byte aligned");
  if (ldx < K || (ldx * 2) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ldx must be >= K with ldx*2 % 16 == 0");
  if (!aligned16(x) || !aligned16(act_packed) || !aligned16(act_scales))
    return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  if ((reinterpret_cast<uintptr_t>(act_packed) & 255u) != 0)
    return fail(COMET_ERR_MISALIGNED, "act_packed must be 256-byte aligned");
  st = check_device();
  if (st != COMET_OK) return st;
  TagMask mask = mask_of(tags_host, K / kBlockK);
  int launches = 0;
  cudaError_t e = perm_dev
      ? launch_quantize_perm(x, xdt == COMET_BF16, M, K, ldx, mask, perm_dev, act_packed, act_scales,
                             static_cast<cudaStream_t>(stream), &launches)
      : launch_quantize(x, xdt == COMET_BF16, M, K, ldx, mask, act_packed, act_scales,
                        static_cast<cudaStream_t>(stream), &launches);
  if (e != cudaSuccess) return cuda_status(e, "quantize launch");
  g_launches = launches;
  return COMET_OK;
}

size_t comet_weight_packed_bytes(int64_t N, int64_t K) {
  if (check_n(N) != COMET_OK || check_mk(1, K) != COMET_OK) return 0;
  return (size_t)N * (size_t)K / 2;
}

comet_status_t comet_pack_weight(const int8_t* w_codes_dev, int64_t N, int64_t K, void* w_packed,
                                 void* stream) {
  g_launches = 0;
  comet_status_t st = check_n(N);
  if (st != COMET_OK) return st;
  st = check_mk(1, K);
  if (st != COMET_OK) return st;
  if (!w_codes_dev || !w_packed) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (!aligned16(w_codes_dev) || !aligned16(w_packed)) return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  st = check_device();
  if (st != COMET_OK) return st;
  cudaError_t e = launch_pack_weight(w_codes_dev, N, K, w_packed, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_status(e, "pack launch");
  g_launches = 1;
  return COMET_OK;
}

comet_status_t comet_pack_weight_perm(const int8_t* w_codes_dev, int64_t N, int64_t K,
                                      const int32_t* perm_dev, void* w_packed, void* stream) {
  if (!perm_dev) return comet_pack_weight(w_codes_dev, N, K, w_packed, stream);
  g_launches = 0;
  comet_status_t st = check_n(N);
  if (st != COMET_OK) return st;
  st = check_mk(1, K);
  if (st != COMET_OK) return st;
  if (!w_codes_dev || !w_packed) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (!aligned16(w_codes_dev) || !aligned16(w_packed) || !aligned16(perm_dev))
    return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  st = check_device();
  if (st != COMET_OK) return st;
  cudaError_t e = launch_pack_weight_perm(w_codes_dev, N, K, perm_dev, w_packed, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_status(e, "pack launch");
  g_launches = 1;
  return COMET_OK;
}

comet_status_t comet_channel_amax(const void* x, comet_dtype_t xdt, int64_t M, int64_t K,
                                  int64_t ldx, float* amax_dev, void* stream) {
  g_launches = 0;
  comet_status_t st = check_mk(M, K);
  if (st != COMET_OK) return st;
  if (!x || !amax_dev) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (xdt != COMET_F16 && xdt != COMET_BF16) return fail(COMET_ERR_INVALID_ARG, "xdt must be COMET_F16 or COMET_BF16");
  if (ldx < K || (ldx * 2) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ldx must be >= K with ldx*2 % 16 == 0");
  if (!aligned16(x) || !aligned16(amax_dev)) return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  st = check_device();
  if (st != COMET_OK) return st;
  cudaError_t e = launch_channel_amax(x, xdt == COMET_BF16, M, K, ldx, amax_dev, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_status(e, "channel amax launch");
  g_launches = 1;
  return COMET_OK;
}

static comet_status_t check_kv4(int64_t T, int64_t C, int group) {
  if (T < 1 || T > INT32_MAX) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "T must be in [1, 2^31-1]");
  if (C < 64 || C % 64 != 0 || C > (int64_t)1 << 20) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "C must be a positive multiple of 64");
  if (group != 32 && group != 64 && group != 128 && group != 256)
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "group must be 32, 64, 128 or 256");
  if (ceil_div(T, group) > 65535) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "too many token groups (T / group > 65535)");
  return COMET_OK;
}

comet_status_t comet_kv4_quantize(const void* kv, comet_dtype_t dt, int64_t T, int64_t C,
                                  int64_t ld, int group, uint8_t* kv4_codes, float* kv4_scales,
                                  float* kv4_mins, void* stream) {
  g_launches = 0;
  comet_status_t st = check_kv4(T, C, group);
  if (st != COMET_OK) return st;
  if (!kv || !kv4_codes || !kv4_scales || !kv4_mins) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (dt != COMET_F16 && dt != COMET_BF16) return fail(COMET_ERR_INVALID_ARG, "dt must be COMET_F16 or COMET_BF16");
  if (ld < C || (ld * 2) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ld must be >= C with ld*2 % 16 == 0");
  if (!aligned16(kv) || !aligned16(kv4_codes) || !aligned16(kv4_scales) || !aligned16(kv4_mins))
    return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  st = check_device();
  if (st != COMET_OK) return st;
  cudaError_t e = launch_kv4_quantize(kv, dt == COMET_BF16, T, C, ld, group, kv4_codes, kv4_scales,
                                      kv4_mins, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_status(e, "kv4 quantize launch");
  g_launches = 1;
  return COMET_OK;
}

comet_status_t comet_kv4_dequantize(const uint8_t* kv4_codes, const float* kv4_scales,
                                    const float* kv4_mins, int64_t T, int64_t C, int group,
                                    void* out, comet_dtype_t odt, int64_t ldo, void* stream) {
  g_launches = 0;
  comet_status_t st = check_kv4(T, C, group);
  if (st != COMET_OK) return st;
  if (!kv4_codes || !kv4_scales || !kv4_mins || !out) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (odt != COMET_F16 && odt != COMET_BF16) return fail(COMET_ERR_INVALID_ARG, "odt must be COMET_F16 or COMET_BF16");
  if (ldo < C || (ldo * 2) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ldo must be >= C with ldo*2 % 16 == 0");
  if (!aligned16(kv4_codes) || !aligned16(kv4_scales) || !aligned16(kv4_mins) || !aligned16(out))
    return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  st = check_device();
  if (st != COMET_OK) return st;
  cudaError_t e = launch_kv4_dequantize(kv4_codes, kv4_scales, kv4_mins, T, C, group, out,
                                        odt == COMET_BF16, ldo, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_status(e, "kv4 dequantize launch");
  g_launches = 1;
  return COMET_OK;
}

void comet_sched_config_default(comet_sched_config* cfg) {
  if (!cfg) return;
  memset(cfg, 0, sizeof(*cfg));
  cfg->tile_n = 0;
  cfg->num_sms = 0;
  cfg->split_mode = -1;
  cfg->cost_int4 = 1.0f;
  cfg->cost_int8 = 1.0f;
  cfg->stages = 0;
  cfg->device_plan = 1;
  cfg->orientation = 0;
}

comet_status_t comet_plan_create(int64_t M, int64_t N, int64_t K, const uint8_t* tags_host,
                                 const comet_sched_config* cfg_in, comet_plan_t* out,
                                 size_t* workspace_bytes) {
  if (!out || !tags_host) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  *out = nullptr;
  comet_status_t st = check_mk(M, K);
  if (st != COMET_OK) return st;
  st = check_n(N);
  if (st != COMET_OK) return st;
  comet_sched_config cfg;
  if (cfg_in) cfg = *cfg_in;
  else comet_sched_config_default(&cfg);
  if (cfg.split_mode < -1 || cfg.split_mode > 3) return fail(COMET_ERR_INVALID_ARG, "split_mode must be -1, 0, 1, 2 or 3");
  if (cfg.cost_int4 < 0 || cfg.cost_int8 < 0) return fail(COMET_ERR_INVALID_ARG, "costs must be >= 0");
  if (cfg.orientation < 0 || cfg.orientation > 4) return fail(COMET_ERR_INVALID_ARG, "orientation must be 0..4");
  if (cfg.num_sms <= 0) {
    if (!cfg.device_plan) return fail(COMET_ERR_INVALID_ARG, "a host-only plan needs an explicit num_sms");
    int sms = 0;
    st = check_device(&sms);
    if (st != COMET_OK) return st;
    cfg.num_sms = sms;
  } else if (cfg.device_plan) {
    int sms = 0;
    st = check_device(&sms);
    if (st != COMET_OK) return st;
    if (cfg.num_sms > sms) return fail(COMET_ERR_INVALID_ARG, "num_sms exceeds the device's SM count (persistent CTAs must be co-resident)");
  }
  comet_plan_s* h = new (std::nothrow) comet_plan_s();
  if (!h) return fail(COMET_ERR_INVALID_ARG, "out of host memory");
  Plan& p = h->p;
  p.M = M; p.N = N; p.K = K;
  p.tags.assign(tags_host, tags_host + K / kBlockK);
  p.mask = mask_of(tags_host, K / kBlockK);
  st = build_plan(p, cfg);
  if (st != COMET_OK) { delete h; return st; }
  p.stages = gemm_stages(p);
  if (cfg.stages != 0 && cfg.stages != p.stages) {
    const std::string msg = "stages: the kernel this plan runs is compiled with a ring depth of " +
                            std::to_string(p.stages) + " (0 = auto)";
    delete h;
    return fail(COMET_ERR_INVALID_ARG, msg);
  }
  if (cfg.device_plan) {
    // the persistent grid must be co-resident (stream-K owners wait for other units' partials):
    // clamp it to what the occupancy calculator admits (e.g. CTA-pair clusters when a GPC has
    // an odd number of SMs)
    int sms = 0;
    check_device(&sms);
    const int units = max_coresident_units(p, sms);
    if (units <= 0) { delete h; return fail(COMET_ERR_CUDA, "occupancy query of the GEMM kernel failed"); }
    if (p.num_ctas > units) {
      comet_sched_config c2 = cfg;
      c2.num_sms = p.orientation == 3 ? 2 * units : units;
      c2.orientation = p.orientation;
      st = build_plan(p, c2);
      if (st != COMET_OK) { delete h; return st; }
    }
  }
  if (cfg.device_plan) {
    cudaGetDevice(&p.device);
    cudaError_t e = cudaMalloc(&p.d_cta_begin, p.cta_begin.size() * sizeof(int32_t));
    if (e == cudaSuccess) e = cudaMalloc(&p.d_items, std::max<size_t>(1, p.items.size()) * sizeof(WorkItem));
    if (e == cudaSuccess) e = cudaMemcpy(p.d_cta_begin, p.cta_begin.data(), p.cta_begin.size() * sizeof(int32_t), cudaMemcpyHostToDevice);
    if (e == cudaSuccess && !p.items.empty())
      e = cudaMemcpy(p.d_items, p.items.data(), p.items.size() * sizeof(WorkItem), cudaMemcpyHostToDevice);
    if (e == cudaSuccess) e = cudaMalloc(&p.d_fix, std::max<size_t>(2, p.fix_info.size()) * sizeof(int32_t));
    if (e == cudaSuccess && !p.fix_info.empty())
      e = cudaMemcpy(p.d_fix, p.fix_info.data(), p.fix_info.size() * sizeof(int32_t), cudaMemcpyHostToDevice);
    if (e != cudaSuccess) {
      if (p.d_cta_begin) cudaFree(p.d_cta_begin);
      if (p.d_items) cudaFree(p.d_items);
      if (p.d_fix) cudaFree(p.d_fix);
      delete h;
      return cuda_status(e, "plan upload");
    }
  }
  if (workspace_bytes) *workspace_bytes = p.ws_bytes;
  h->cfg = cfg;
  *out = h;
  return COMET_OK;
}

comet_status_t comet_plan_destroy(comet_plan_t plan) {
  if (!plan) return COMET_OK;
  if (plan->chunk) comet_plan_destroy(plan->chunk);
  if (plan->tail) comet_plan_destroy(plan->tail);
  for (cudaEvent_t e : plan->ev) cudaEventDestroy(e);
  // s_h2d / s_d2h are the device's shared copy streams (copy_streams), not owned by the plan
  if (plan->p.d_cta_begin) cudaFree(plan->p.d_cta_begin);
  if (plan->p.d_items) cudaFree(plan->p.d_items);
  if (plan->p.d_fix) cudaFree(plan->p.d_fix);
  delete plan;
  return COMET_OK;
}

comet_status_t comet_plan_info(comet_plan_t plan, comet_plan_info_t* info) {
  if (!plan || !info) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  const Plan& p = plan->p;
  info->M = p.M; info->N = p.N; info->K = p.K;
  info->tile_n = p.tile_n; info->num_ctas = p.num_ctas; info->split_mode = p.split_mode;
  info->stages = p.stages;
  info->orientation = p.orientation;
  info->tile_w = p.tile_w;
  info->n_tiles = p.n_tiles;
  info->n_items = (int64_t)p.items.size();
  info->n_split_tiles = p.n_split_tiles;
  info->max_cta_cost = p.max_cost;
  info->mean_cta_cost = p.mean_cost;
  return COMET_OK;
}

comet_status_t comet_plan_describe(comet_plan_t plan, int32_t* items, int64_t max_items, int64_t* n_items) {
  if (!plan || !n_items) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  const Plan& p = plan->p;
  int64_t n = 0;
  for (int c = 0; c < p.num_ctas; ++c) {
    for (int i = p.cta_begin[c]; i < p.cta_begin[c + 1]; ++i) {
      if (items && n < max_items) {
        items[4 * n + 0] = c;
        items[4 * n + 1] = p.items[i].tile;
        items[4 * n + 2] = p.items[i].kb_begin;
        items[4 * n + 3] = p.items[i].kb_end;
      }
      ++n;
    }
  }
  *n_items = items ? std::min(n, max_items) : n;
  return COMET_OK;
}

comet_status_t comet_w4ax_gemm(comet_plan_t plan, const void* act_packed, const float* act_scales,
                               const void* w_packed, const float* w_scales, void* y,
                               comet_dtype_t ydt, int64_t ldy, int32_t* debug_acc,
                               int32_t* debug_acc_blocks, void* workspace, size_t ws_bytes,
                               void* stream) {
  g_launches = 0;
  if (!plan || !act_packed || !act_scales || !w_packed || !w_scales || !y)
    return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  Plan& p = plan->p;
  if (ydt != COMET_F16 && ydt != COMET_BF16 && ydt != COMET_F32) return fail(COMET_ERR_INVALID_ARG, "bad ydt");
  const int esz = ydt == COMET_F32 ? 4 : 2;
  if (ldy < p.N || (ldy * esz) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ldy must be >= N with ldy*sizeof(y) % 16 == 0");
  if ((reinterpret_cast<uintptr_t>(act_packed) & 255u) != 0) return fail(COMET_ERR_MISALIGNED, "act_packed must be 256-byte aligned");
  if (!aligned16(act_scales) || !aligned16(w_packed) || !aligned16(w_scales) || !aligned16(y) ||
      (debug_acc && !aligned16(debug_acc)) || (debug_acc_blocks && !aligned16(debug_acc_blocks)) ||
      (workspace && !aligned16(workspace)))
    return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  comet_status_t st = check_device();
  if (st != COMET_OK) return st;
  int launches = 0;
  st = launch_gemm(p, act_packed, act_scales, w_packed, w_scales, y, ydt, ldy, debug_acc,
                   debug_acc_blocks, workspace, ws_bytes, static_cast<cudaStream_t>(stream), &launches);
  g_launches = launches;
  return st;
}

comet_status_t comet_w4ax_linear(comet_plan_t plan, const void* x, comet_dtype_t xdt, int64_t ldx,
                                 const void* w_packed, const float* w_scales, void* y,
                                 comet_dtype_t ydt, int64_t ldy, void* workspace, size_t ws_bytes,
                                 void* stream) {
  g_launches = 0;
  if (!plan || !x || !w_packed || !w_scales || !y) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  Plan& p = plan->p;
  if (xdt != COMET_F16 && xdt != COMET_BF16) return fail(COMET_ERR_INVALID_ARG, "x must be F16 or BF16");
  if (ydt != COMET_F16 && ydt != COMET_BF16 && ydt != COMET_F32) return fail(COMET_ERR_INVALID_ARG, "bad ydt");
  if (ldx < p.K || (ldx * 2) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ldx must be >= K with ldx*2 % 16 == 0");
  const int esz = ydt == COMET_F32 ? 4 : 2;
  if (ldy < p.N || (ldy * esz) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ldy must be >= N with ldy*sizeof(y) % 16 == 0");
  if (!aligned16(x) || !aligned16(w_packed) || !aligned16(w_scales) || !aligned16(y) ||
      (workspace && !aligned16(workspace)))
    return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  comet_status_t st = check_device();
  if (st != COMET_OK) return st;
  const FusedX fx{x, ldx, xdt == COMET_BF16};
  int launches = 0;
  st = launch_gemm(p, nullptr, nullptr, w_packed, w_scales, y, ydt, ldy, nullptr, nullptr, workspace,
                   ws_bytes, static_cast<cudaStream_t>(stream), &launches, false, nullptr, &fx);
  g_launches = launches;
  return st;
}

comet_status_t comet_w4ax_gemm_grouped(comet_plan_t plan, const void* act_packed, const float* act_scales,
                                       const void* w_packed, const float* w_scales_grouped, void* y,
                                       comet_dtype_t ydt, int64_t ldy, int32_t* debug_acc,
                                       void* workspace, size_t ws_bytes, void* stream) {
  g_launches = 0;
  if (!plan || !act_packed || !act_scales || !w_packed || !w_scales_grouped || !y)
    return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  Plan& p = plan->p;
  if (ydt != COMET_F16 && ydt != COMET_BF16 && ydt != COMET_F32) return fail(COMET_ERR_INVALID_ARG, "bad ydt");
  const int esz = ydt == COMET_F32 ? 4 : 2;
  if (ldy < p.N || (ldy * esz) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ldy must be >= N with ldy*sizeof(y) % 16 == 0");
  if ((reinterpret_cast<uintptr_t>(act_packed) & 255u) != 0) return fail(COMET_ERR_MISALIGNED, "act_packed must be 256-byte aligned");
  if (!aligned16(act_scales) || !aligned16(w_packed) || !aligned16(w_scales_grouped) || !aligned16(y) ||
      (debug_acc && !aligned16(debug_acc)) || (workspace && !aligned16(workspace)))
    return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  if (p.orientation != 1 && !(p.orientation == 3 && p.tile_w == 256))
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "group-wise weight scales run on orientation 1 or on the 256-wide pair kernel (orientation 3)");
  comet_status_t st = check_device();
  if (st != COMET_OK) return st;
  int launches = 0;
  st = launch_gemm(p, act_packed, act_scales, w_packed, w_scales_grouped, y, ydt, ldy, debug_acc, nullptr,
                   workspace, ws_bytes, static_cast<cudaStream_t>(stream), &launches, true);
  g_launches = launches;
  return st;
}

static int64_t rs_rows_per_rank(int64_t M, int world) { return ceil_div(M, world); }

size_t comet_rs_recv_bytes(int64_t M, int64_t N, int world) {
  if (M < 1 || N < 1 || world < 1 || world > 8) return 0;
  return (size_t)world * (size_t)rs_rows_per_rank(M, world) * (size_t)N * sizeof(float);
}

comet_status_t comet_w4ax_gemm_rs(comet_plan_t plan, const void* act_packed, const float* act_scales,
                                  const void* w_packed, const float* w_scales, float* const* recv_bufs_host,
                                  int world, int rank, void* workspace, size_t ws_bytes, void* stream) {
  g_launches = 0;
  if (!plan || !act_packed || !act_scales || !w_packed || !w_scales || !recv_bufs_host)
    return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (world < 1 || world > 8 || rank < 0 || rank >= world) return fail(COMET_ERR_INVALID_ARG, "world must be 1..8 and 0 <= rank < world");
  Plan& p = plan->p;
  if (p.orientation != 3 || p.tile_w != 256)
    return fail(COMET_ERR_UNSUPPORTED_SHAPE, "the fused reduce-scatter runs on the 256-wide CTA-pair prefill kernel (plan orientation 3, tile_w 256)");
  RsArgs rs{};
  rs.world = world;
  rs.rank = rank;
  rs.ms = rs_rows_per_rank(p.M, world);
  for (int i = 0; i < world; ++i) {
    if (!recv_bufs_host[i]) return fail(COMET_ERR_INVALID_ARG, "NULL receive buffer");
    if (!aligned16(recv_bufs_host[i])) return fail(COMET_ERR_MISALIGNED, "receive buffers must be 16-byte aligned");
    rs.dst[i] = recv_bufs_host[i];
  }
  if ((reinterpret_cast<uintptr_t>(act_packed) & 255u) != 0) return fail(COMET_ERR_MISALIGNED, "act_packed must be 256-byte aligned");
  if (!aligned16(act_scales) || !aligned16(w_packed) || !aligned16(w_scales) || (workspace && !aligned16(workspace)))
    return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  comet_status_t st = check_device();
  if (st != COMET_OK) return st;
  int launches = 0;
  // y is never written on this path (the epilogue stores to the receive buffers); the local
  // receive buffer stands in for the output tensor map
  st = launch_gemm(p, act_packed, act_scales, w_packed, w_scales, recv_bufs_host[rank], COMET_F32, p.N, nullptr,
                   nullptr, workspace, ws_bytes, static_cast<cudaStream_t>(stream), &launches, false, &rs);
  g_launches = launches;
  return st;
}

comet_status_t comet_rs_reduce(const float* recv_local, int world, int rank, int64_t M, int64_t N, void* y,
                               comet_dtype_t ydt, int64_t ldy, void* stream) {
  g_launches = 0;
  if (!recv_local || !y) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (world < 1 || world > 8 || rank < 0 || rank >= world) return fail(COMET_ERR_INVALID_ARG, "world must be 1..8 and 0 <= rank < world");
  if (N % 4 != 0) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "N must be a multiple of 4");
  if (ydt != COMET_F16 && ydt != COMET_BF16 && ydt != COMET_F32) return fail(COMET_ERR_INVALID_ARG, "bad ydt");
  const int esz = ydt == COMET_F32 ? 4 : 2;
  if (ldy < N || (ldy * esz) % 16 != 0) return fail(COMET_ERR_MISALIGNED, "ldy must be >= N with ldy*sizeof(y) % 16 == 0");
  if (!aligned16(recv_local) || !aligned16(y)) return fail(COMET_ERR_MISALIGNED, "device pointers must be 16-byte aligned");
  const int64_t ms = rs_rows_per_rank(M, world);
  const int64_t rows = std::max<int64_t>(0, std::min<int64_t>(ms, M - (int64_t)rank * ms));
  comet_status_t st = check_device();
  if (st != COMET_OK) return st;
  // the slots of the source ranks are [src][ms][N]; this rank owns `rows` of them
  cudaError_t e = launch_rs_reduce(recv_local, world, rows, ms, N, y, (int)ydt, ldy, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return cuda_status(e, "reduce launch");
  g_launches = 1;
  return COMET_OK;
}

// Pipelined host path: chunks of kLinChunk token rows once M >= 2 kLinChunk.
static constexpr int64_t kLinChunk = 1024;

static int64_t lin_chunks(const Plan& p) { return p.M >= 2 * kLinChunk ? ceil_div(p.M, kLinChunk) : 1; }

// Sub-plans of the pipelined path (device plans, same scheduler configuration as the parent).
static comet_status_t ensure_subplans(comet_plan_t plan) {
  const Plan& p = plan->p;
  if (lin_chunks(p) == 1 || plan->chunk) return COMET_OK;
  comet_sched_config cfg = plan->cfg;
  cfg.device_plan = 1;
  comet_status_t st = comet_plan_create(kLinChunk, p.N, p.K, p.tags.data(), &cfg, &plan->chunk, nullptr);
  if (st != COMET_OK) return st;
  const int64_t rem = p.M % kLinChunk;
  if (rem) {
    st = comet_plan_create(rem, p.N, p.K, p.tags.data(), &cfg, &plan->tail, nullptr);
    if (st != COMET_OK) return st;
  }
  return COMET_OK;
}

struct LinLayout {
  size_t x_off, act_off, sc_off, y_off, ws_chunk_off, ws_tail_off, total;
};

// scratch: [x: M x K (16-bit)] [act packed: one chunk] [scales: one chunk] [y: M x N]
//          [fix-up workspace of the chunk plan] [... of the tail plan]
static LinLayout lin_layout(comet_plan_t plan, comet_dtype_t ydt) {
  const Plan& p = plan->p;
  const int64_t mc = lin_chunks(p) == 1 ? p.M : kLinChunk;
  comet_act_layout_t L;
  act_layout(mc, p.K, &L);
  LinLayout o;
  size_t off = 0;
  o.x_off = off;
  off += (size_t)round_up(p.M * p.K * 2, 256);
  o.act_off = off;
  off += L.total_bytes;
  o.sc_off = off;
  off += (size_t)round_up((int64_t)(L.nb * L.Mp * 4), 256);
  o.y_off = off;
  off += (size_t)round_up(p.M * p.N * (ydt == COMET_F32 ? 4 : 2), 256);
  o.ws_chunk_off = off;
  if (plan->chunk) off += (size_t)round_up((int64_t)plan->chunk->p.ws_bytes, 256);
  o.ws_tail_off = off;
  if (plan->tail) off += (size_t)round_up((int64_t)plan->tail->p.ws_bytes, 256);
  o.total = off;
  return o;
}

size_t comet_linear_scratch_bytes(comet_plan_t plan, comet_dtype_t xdt, comet_dtype_t ydt) {
  (void)xdt;
  if (!plan) return 0;
  if (ensure_subplans(plan) != COMET_OK) return 0;
  return lin_layout(plan, ydt).total;
}

// One host-to-device and one device-to-host copy stream per device, shared by every plan's
// host pipeline: consecutive calls (e.g. a model's layers issued back to back) then upload and
// download in call order at the full PCIe rate of each direction, instead of splitting it over
// several concurrent per-plan streams (which delays the first layer's downloads).
static cudaError_t copy_streams(cudaStream_t* h2d, cudaStream_t* d2h) {
  static std::mutex mu;
  static cudaStream_t streams[64][2] = {};
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  std::lock_guard<std::mutex> lock(mu);
  if (!streams[dev][0]) {
    e = cudaStreamCreateWithFlags(&streams[dev][0], cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&streams[dev][1], cudaStreamNonBlocking);
    if (e != cudaSuccess) return e;
  }
  *h2d = streams[dev][0];
  *d2h = streams[dev][1];
  return cudaSuccess;
}

static comet_status_t linear_host(comet_plan_t plan, const void* x_host, comet_dtype_t xdt,
                                  const void* w_packed, const float* w_scales, void* y_host,
                                  comet_dtype_t ydt, void* scratch, size_t scratch_bytes,
                                  void* workspace, size_t ws_bytes, void* stream, bool blocking) {
  if (!plan || !x_host || !y_host || !scratch) return fail(COMET_ERR_INVALID_ARG, "NULL pointer argument");
  if (xdt != COMET_F16 && xdt != COMET_BF16) return fail(COMET_ERR_INVALID_ARG, "xdt must be F16 or BF16");
  Plan& p = plan->p;
  comet_status_t st = ensure_subplans(plan);
  if (st != COMET_OK) return st;
  const LinLayout lay = lin_layout(plan, ydt);
  if (scratch_bytes < lay.total) return fail(COMET_ERR_WORKSPACE_TOO_SMALL, "scratch smaller than comet_linear_scratch_bytes");
  if ((reinterpret_cast<uintptr_t>(scratch) & 255u) != 0) return fail(COMET_ERR_MISALIGNED, "scratch must be 256-byte aligned");
  uint8_t* s = static_cast<uint8_t*>(scratch);
  cudaStream_t cs = static_cast<cudaStream_t>(stream);
  const size_t esz = ydt == COMET_F32 ? 4 : 2;
  const int64_t nch = lin_chunks(p);
  cudaError_t e;
  if (nch == 1) {
    // one chunk: H2D, quantise, GEMM, D2H in order on `stream`
    e = cudaMemcpyAsync(s + lay.x_off, x_host, (size_t)(p.M * p.K * 2), cudaMemcpyHostToDevice, cs);
    if (e != cudaSuccess) return cuda_status(e, "H2D copy");
    st = comet_quantize_act(s + lay.x_off, xdt, p.M, p.K, p.K, p.tags.data(), nullptr, s + lay.act_off,
                            reinterpret_cast<float*>(s + lay.sc_off), stream);
    if (st != COMET_OK) return st;
    const int l1 = g_launches;
    st = comet_w4ax_gemm(plan, s + lay.act_off, reinterpret_cast<float*>(s + lay.sc_off), w_packed, w_scales,
                         s + lay.y_off, ydt, p.N, nullptr, nullptr, workspace, ws_bytes, stream);
    if (st != COMET_OK) return st;
    const int l2 = g_launches;
    e = cudaMemcpyAsync(y_host, s + lay.y_off, (size_t)(p.M * p.N) * esz, cudaMemcpyDeviceToHost, cs);
    if (e != cudaSuccess) return cuda_status(e, "D2H copy");
    // completion event of this call's download: comet_linear_host_wait blocks on it
    if (plan->ev.empty()) {
      cudaEvent_t ev;
      e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
      if (e != cudaSuccess) return cuda_status(e, "event create");
      plan->ev.push_back(ev);
    }
    e = cudaEventRecord(plan->ev[0], cs);
    if (e != cudaSuccess) return cuda_status(e, "event record");
    plan->prev_call = true;
    if (blocking) {
      e = cudaEventSynchronize(plan->ev[0]);
      if (e != cudaSuccess) return cuda_status(e, "D2H synchronize");
    }
    g_launches = l1 + l2;
    return COMET_OK;
  }
  // pipelined.  Dependencies: chunk c's quantise + GEMM (on `stream`, so after the caller's prior
  // work) wait for its H2D; its D2H waits for its GEMM.  Across calls with this plan: the H2D
  // copies wait for the previous call's last quantise (the last reader of the scratch x region)
  // and the first GEMM waits for the previous call's last D2H (the last reader of scratch y).
  // Nothing else orders the copy streams, so one call's uploads overlap the previous call's
  // downloads and compute.
  if (!plan->s_h2d) {
    e = copy_streams(&plan->s_h2d, &plan->s_d2h);
    if (e != cudaSuccess) return cuda_status(e, "copy stream create");
  }
  while ((int64_t)plan->ev.size() < 3 * nch + 2) {
    cudaEvent_t ev;
    e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_status(e, "event create");
    plan->ev.push_back(ev);
  }
  cudaEvent_t ev_quant_last = plan->ev[3 * nch], ev_d2h_last = plan->ev[3 * nch + 1];
  // zero the sub-plans' stream-K flag workspace the first time this scratch is used (flags are
  // compared with process-wide launch epochs, which start at 1)
  if (plan->ws_zeroed != scratch) {
    e = cudaMemsetAsync(s + lay.ws_chunk_off, 0, lay.total - lay.ws_chunk_off, cs);
    if (e != cudaSuccess) return cuda_status(e, "workspace clear");
    plan->ws_zeroed = scratch;
  }
  if (plan->prev_call) {
    e = cudaStreamWaitEvent(plan->s_h2d, ev_quant_last, 0);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, ev_d2h_last, 0);
    if (e != cudaSuccess) return cuda_status(e, "stream ordering");
  }
  int launches = 0;
  for (int64_t c = 0; c < nch; ++c) {
    const int64_t m0 = c * kLinChunk, rows = std::min<int64_t>(kLinChunk, p.M - m0);
    comet_plan_t sub = rows == kLinChunk ? plan->chunk : plan->tail;
    uint8_t* ws = s + (rows == kLinChunk ? lay.ws_chunk_off : lay.ws_tail_off);
    cudaEvent_t e_h2d = plan->ev[3 * c], e_comp = plan->ev[3 * c + 1];
    e = cudaMemcpyAsync(s + lay.x_off + (size_t)(m0 * p.K * 2), static_cast<const uint8_t*>(x_host) + (size_t)(m0 * p.K * 2),
                        (size_t)(rows * p.K * 2), cudaMemcpyHostToDevice, plan->s_h2d);
    if (e == cudaSuccess) e = cudaEventRecord(e_h2d, plan->s_h2d);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, e_h2d, 0);
    if (e != cudaSuccess) return cuda_status(e, "H2D copy");
    st = comet_quantize_act(s + lay.x_off + (size_t)(m0 * p.K * 2), xdt, rows, p.K, p.K, p.tags.data(), nullptr,
                            s + lay.act_off, reinterpret_cast<float*>(s + lay.sc_off), stream);
    if (st != COMET_OK) return st;
    launches += g_launches;
    if (c == nch - 1) {
      e = cudaEventRecord(ev_quant_last, cs);
      if (e != cudaSuccess) return cuda_status(e, "event record");
    }
    st = comet_w4ax_gemm(sub, s + lay.act_off, reinterpret_cast<float*>(s + lay.sc_off), w_packed, w_scales,
                         s + lay.y_off + (size_t)(m0 * p.N) * esz, ydt, p.N, nullptr, nullptr, ws,
                         sub->p.ws_bytes, stream);
    if (st != COMET_OK) return st;
    launches += g_launches;
    e = cudaEventRecord(e_comp, cs);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(plan->s_d2h, e_comp, 0);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(static_cast<uint8_t*>(y_host) + (size_t)(m0 * p.N) * esz, s + lay.y_off + (size_t)(m0 * p.N) * esz,
                          (size_t)(rows * p.N) * esz, cudaMemcpyDeviceToHost, plan->s_d2h);
    if (e != cudaSuccess) return cuda_status(e, "D2H copy");
  }
  e = cudaEventRecord(ev_d2h_last, plan->s_d2h);
  if (e != cudaSuccess) return cuda_status(e, "event record");
  plan->prev_call = true;
  if (blocking) {
    e = cudaEventSynchronize(ev_d2h_last);
    if (e != cudaSuccess) return cuda_status(e, "D2H synchronize");
  }
  g_launches = launches;
  return COMET_OK;
}

comet_status_t comet_linear_host_wait(comet_plan_t plan) {
  if (!plan) return fail(COMET_ERR_INVALID_ARG, "NULL plan");
  if (!plan->prev_call) return COMET_OK;
  const int64_t nch = lin_chunks(plan->p);
  cudaError_t e = cudaEventSynchronize(plan->ev[nch == 1 ? 0 : 3 * nch + 1]);
  if (e != cudaSuccess) return cuda_status(e, "D2H synchronize");
  return COMET_OK;
}

comet_status_t comet_w4ax_linear_host(comet_plan_t plan, const void* x_host, comet_dtype_t xdt,
                                      const void* w_packed, const float* w_scales, void* y_host,
                                      comet_dtype_t ydt, void* scratch, size_t scratch_bytes,
                                      void* workspace, size_t ws_bytes, void* stream) {
  return linear_host(plan, x_host, xdt, w_packed, w_scales, y_host, ydt, scratch, scratch_bytes, workspace,
                     ws_bytes, stream, true);
}

comet_status_t comet_w4ax_linear_host_async(comet_plan_t plan, const void* x_host, comet_dtype_t xdt,
                                            const void* w_packed, const float* w_scales, void* y_host,
                                            comet_dtype_t ydt, void* scratch, size_t scratch_bytes,
                                            void* workspace, size_t ws_bytes, void* stream) {
  return linear_host(plan, x_host, xdt, w_packed, w_scales, y_host, ydt, scratch, scratch_bytes, workspace,
                     ws_bytes, stream, false);
}

}  // extern "C"
