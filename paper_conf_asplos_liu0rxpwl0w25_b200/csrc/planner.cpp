// planner.cpp -- host-side tile scheduler ("fine-grained SM scheduling").
//
// Scheduling unit = (output tile, 128-channel K-block): the paper's 128x128x128 "tile"
// (P:L212).  A unit costs cost_int8 or cost_int4 by its block's tag (on the paper's A100 the
// INT4 tensor core is 2x faster; on B200 both precisions run at the same tensor rate,
// so the default is 1:1).  Every persistent CTA walks its own work list; the only inter-CTA
// synchronisation is the fix-up of tiles whose units landed on several CTAs, before
// write-back (barrier minimisation).
//
//   split_mode 2  naive (Fig. 8b/c): units dealt round-robin in unit order.
//   split_mode 3  unit remapping (Fig. 8d): units longest-first onto the least-loaded
//                 CTA (LPT), balancing INT4 against INT8 units.
//   split_mode 0  whole-tile remapping: whole tiles onto the least-loaded CTA; no fix-up.
//   split_mode 1  tile decomposition (Fig. 8e; stream-K [42]): all but the last
//                 1-2 waves run as whole tiles, the remaining tiles' units are cut into P
//                 contiguous ranges with the smallest possible maximum cost.
// Units of one tile on one CTA are merged into contiguous K-ranges ("segments").  A tile with
// several segments is finished by the CTA holding its K-block 0 (the owner), which adds the
// other segments' FP32 partials in K order (deterministic).  Every CTA runs its non-owner
// segments before anything that can wait, so waits never form a cycle.
#include <algorithm>
#include <cmath>
#include <map>
#include <numeric>
#include <queue>
#include "internal.h"

namespace comet {

static int auto_tile_n(int64_t M) {
  if (M <= 16) return 16;
  if (M <= 32) return 32;
  if (M <= 64) return 64;
  return 128;
}

static bool valid_tile_n(int nt) {
  return nt == 16 || nt == 32 || nt == 64 || nt == 128;
}

// Smallest max-part cost when cutting `cost` (a sequence) into at most P contiguous parts;
// returns the cut positions (first unit of each part, P+1 entries).
static std::vector<int64_t> best_contiguous_cuts(const std::vector<double>& cost, int P) {
  const int64_t n = (int64_t)cost.size();
  std::vector<int64_t> cut(P + 1, n);
  cut[0] = 0;
  if (n == 0) return cut;
  double lo = *std::max_element(cost.begin(), cost.end());
  double hi = std::accumulate(cost.begin(), cost.end(), 0.0);
  lo = std::max(lo, hi / P);
  auto parts_needed = [&](double cap) {
    int parts = 1;
    double s = 0;
    for (double c : cost) {
      if (s + c > cap + 1e-9) { ++parts; s = c; } else { s += c; }
    }
    return parts;
  };
  for (int iter = 0; iter < 60 && hi - lo > 1e-6; ++iter) {
    const double mid = 0.5 * (lo + hi);
    if (parts_needed(mid) <= P) hi = mid; else lo = mid;
  }
  // greedy cut at capacity `hi`, then spread remaining parts evenly is not needed: greedy
  // with the optimal cap already uses <= P parts.
  int part = 0;
  double s = 0;
  for (int64_t u = 0; u < n; ++u) {
    if (s + cost[u] > hi + 1e-9) { cut[++part] = u; s = 0; }
    s += cost[u];
  }
  for (int p2 = part + 1; p2 <= P; ++p2) cut[p2] = n;
  return cut;
}

comet_status_t build_plan(Plan& p, const comet_sched_config& cfg) {
  p.nb = p.K / kBlockK;
  p.Mp = round_up(p.M, COMET_SCALE_PAD);
  p.orientation = cfg.orientation > 0 ? cfg.orientation : (p.M >= 256 ? 3 : (p.M >= 128 ? 2 : 1));
  // decode on the warp-level path (gemm_v.cu) where it measured faster than the TMEM kernel
  // (tools/gemv_ab.py): M <= 8 with >= 32 MiB of packed weights (LLaMA-3-70B: gate/up M = 1 / 4 / 8
  // 23.3 / 24.0 / 26.7 vs 28.0 / 27.3 / 27.8 us, down 23.6 / 24.6 / 27.6 vs 26.6 / 26.7 / 27.3,
  // qkv 11.7 / 12.1 / 11.9 vs 14.2), or >= 8 MiB when N >= K (LLaMA-2-7B q/k/v/o 7.2 vs 7.5 us,
  // gate/up 9.4 vs 10.5; its down, K = 11008 > N, 10.5-11.0 vs 10.4-10.5, stays on 1)
  bool auto_o4 = false;
  if (cfg.orientation <= 0 && p.M <= 8 &&
      (p.N * p.K / 2 >= (32ll << 20) || (p.N * p.K / 2 >= (8ll << 20) && p.N >= p.K))) {
    int nbr = 0, s = 0;
    auto_o4 = gemv::gemv_pick(p.M, (p.N / 128) * (p.K / kBlockK), (int)(p.K / kBlockK), cfg.num_sms, &nbr, &s) > 0;
    if (auto_o4) p.orientation = 4;
  }
  if (p.orientation == 4) {
    // decode on the warp-level tensor-core path (gemm_v.cu): units (128-row group, K-block),
    // group-major, cut into one contiguous range per CTA (CTA-level stream-K); no work list,
    // the partials go through the workspace
    if (p.M > 8) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "orientation 4 takes M <= 8 tokens");
    p.tile_n = 8;
    p.tile_w = 128;
    p.split_mode = 1;
    p.kgran = 1;
    if (cfg.num_sms <= 0) return fail(COMET_ERR_INVALID_ARG, "num_sms must be resolved before planning");
    p.n_m_tiles = 1;
    p.n_n_tiles = p.N / 128;
    p.n_tiles = p.n_n_tiles;
    const int64_t units = p.n_tiles * p.nb;
    p.num_ctas = gemv::gemv_pick(p.M, units, (int)p.nb, cfg.num_sms, &p.gemv_nbr, &p.gemv_s);
    if (p.num_ctas < 0) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "orientation 4: shape unsupported (a CTA's K range exceeds the activation staging capacity, or more than 64 CTAs share a row group)");
    const int P = p.num_ctas;
    p.max_segments = gemv::gemv_max_segments(units, (int)p.nb, P);
    p.n_split_tiles = 0;                       // groups shared by more than one CTA
    for (int64_t t = 0; t < p.n_tiles; ++t) {
      const int64_t ua = t * p.nb, ub = ua + p.nb - 1;
      if (((ua + 1) * P - 1) / units != ((ub + 1) * P - 1) / units) p.n_split_tiles++;
    }
    p.cta_begin.assign(P + 1, 0);
    p.items.clear();
    p.fix_info.clear();
    p.max_cost = (double)((units + P - 1) / P);
    p.mean_cost = (double)units / P;
    // partial slots [ctas][max_segments][128][8] f32
    p.ws_flags_off = 0;
    p.ws_bytes = ((size_t)P * p.max_segments * 128 * 8 * sizeof(float) + 255) / 256 * 256;
    return COMET_OK;
  }
  if (p.orientation >= 2) {
    p.tile_n = p.orientation == 3 ? 256 : 128;   // tokens per tile = MMA M (CTA pair: 2 x 128)
    p.tile_w = cfg.tile_w > 0 ? cfg.tile_w : (p.orientation == 3 ? 256 : 192);  // weights per tile = MMA N
    if (p.tile_w != 128 && p.tile_w != 160 && p.tile_w != 192 && !(p.tile_w == 256 && p.orientation == 3))
      return fail(COMET_ERR_UNSUPPORTED_SHAPE, "tile_w must be 128, 160 or 192 (or 256 with orientation 3)");
  } else {
    p.tile_n = cfg.tile_n > 0 ? cfg.tile_n : auto_tile_n(p.M);
    p.tile_w = kTileW;
    if (!valid_tile_n(p.tile_n))
      return fail(COMET_ERR_UNSUPPORTED_SHAPE, "tile_n must be one of 16, 32, 64, 128");
  }
  // scheduling units: CTAs, or CTA pairs for the pair kernel
  p.num_ctas = p.orientation == 3 ? cfg.num_sms / 2 : cfg.num_sms;
  if (p.num_ctas <= 0) return fail(COMET_ERR_INVALID_ARG, "num_sms must be resolved before planning (>= 2 for CTA pairs)");
  p.n_m_tiles = ceil_div(p.M, p.tile_n);
  p.n_n_tiles = ceil_div(p.N, p.tile_w);
  p.n_tiles = p.n_m_tiles * p.n_n_tiles;
  const int P = p.num_ctas;
  const int64_t T = p.n_tiles;
  const int nkb = (int)p.nb;
  const double c4 = cfg.cost_int4 > 0 ? cfg.cost_int4 : 1.0;
  const double c8 = cfg.cost_int8 > 0 ? cfg.cost_int8 : 1.0;

  int mode = cfg.split_mode;
  if (mode < 0) {
    const double eff = (double)T / ((double)P * (double)ceil_div(T, P));   // whole-tile efficiency
    mode = eff < 0.92 ? 1 : 0;
  }
  if (mode < 0 || mode > 3) return fail(COMET_ERR_INVALID_ARG, "split_mode must be -1..3");
  p.split_mode = mode;
  // Scheduling granularity: the decode kernel streams 4 K-blocks per pipeline stage at
  // tile_n <= 32, so its stream-K / whole-tile cuts fall on 4-K-block boundaries (a cut
  // elsewhere would load weights another CTA also loads).  The paper's unit-level modes 2/3
  // (Fig. 8) keep single K-blocks.
  const int kgran = (p.orientation == 1 && p.tile_n <= 32 && (mode == 0 || mode == 1)) ? 4 : 1;
  p.kgran = kgran;
  const int nb = (int)ceil_div(nkb, kgran);          // scheduling units per tile
  std::vector<double> ucost(nb, 0.0);
  for (int b = 0; b < nkb; ++b) ucost[b / kgran] += p.tags[b] ? c8 : c4;
  const double tile_cost = std::accumulate(ucost.begin(), ucost.end(), 0.0);

  // ---- assignment: for every CTA an ordered list of (tile, kb) runs
  struct Run { int64_t tile; int kb0, kb1; };
  std::vector<std::vector<Run>> runs(P);
  std::vector<double> load(P, 0.0);
  auto add_unit = [&](int cta, int64_t tile, int kb) {
    auto& r = runs[cta];
    if (!r.empty() && r.back().tile == tile && r.back().kb1 == kb) r.back().kb1 = kb + 1;
    else r.push_back({tile, kb, kb + 1});
    load[cta] += ucost[kb];
  };
  // Tile order for the whole-tile assignments (prefill orientations).  A wave of P concurrent
  // tiles streams its operands along K once; what a wave touches is (#token tiles) x (token
  // tile's codes, M_t x K bytes) + (#weight tiles) x (weight tile, tile_w x K/2 bytes).  When
  // the whole activation matrix fits in L2 (<= 48 MB: every LLaMA layer with K <= 8192 at
  // M = 4096) the natural order -- token tiles fastest, so each wave covers all of them and
  // few weight tiles -- reads everything once.  Otherwise (LLaMA-3-70B down, K = 28672:
  // 117 MB of codes, read 3.5x per launch in the natural order) the tiles are visited in
  // groups of GN weight tiles with every token tile against each group, GN chosen so a wave
  // is a balanced block: GN = sqrt(P * token-tile bytes / weight-tile bytes).  Decode
  // (orientation 1) keeps the natural order.
  std::vector<int64_t> order((size_t)T);
  {
    int64_t gn = p.n_n_tiles;
    const double act_bytes = (double)p.M * (double)p.K;
    if (p.orientation >= 2 && act_bytes > 48.0 * (1 << 20)) {
      const double abytes = (double)p.tile_n * (double)p.K;           // codes per token tile
      const double wbytes = (double)p.tile_w * (double)p.K / 2.0;     // packed weights per tile
      gn = std::max<int64_t>(1, std::min<int64_t>(p.n_n_tiles, (int64_t)std::llround(std::sqrt((double)P * abytes / wbytes))));
    }
    if (gn >= p.n_n_tiles) {
      for (int64_t t = 0; t < T; ++t) order[(size_t)t] = t;         // natural: token tiles fastest
    } else {
      int64_t i = 0;
      for (int64_t g0 = 0; g0 < p.n_n_tiles; g0 += gn)
        for (int64_t m = 0; m < p.n_m_tiles; ++m)
          for (int64_t n = g0; n < std::min(p.n_n_tiles, g0 + gn); ++n) order[(size_t)i++] = n * p.n_m_tiles + m;
    }
  }
  if (mode == 0) {
    using E = std::pair<double, int>;
    std::priority_queue<E, std::vector<E>, std::greater<E>> pq;
    for (int c = 0; c < P; ++c) pq.push({0.0, c});
    for (int64_t ti = 0; ti < T; ++ti) {
      const int64_t t = order[(size_t)ti];
      auto [l, c] = pq.top();
      pq.pop();
      runs[c].push_back({t, 0, nb});
      load[c] += tile_cost;
      pq.push({l + tile_cost, c});
    }
  } else if (mode == 2) {
    int64_t u = 0;
    for (int64_t t = 0; t < T; ++t)
      for (int kb = 0; kb < nb; ++kb, ++u) add_unit((int)(u % P), t, kb);
  } else if (mode == 3) {
    // LPT over units: most expensive first (stable within equal cost: unit order)
    std::vector<int> kb_order(nb);
    std::iota(kb_order.begin(), kb_order.end(), 0);
    std::stable_sort(kb_order.begin(), kb_order.end(), [&](int a, int b) { return ucost[a] > ucost[b]; });
    using E = std::pair<double, int>;
    std::priority_queue<E, std::vector<E>, std::greater<E>> pq;
    for (int c = 0; c < P; ++c) pq.push({0.0, c});
    // visit units grouped by cost class, tile-major inside a class
    std::vector<double> classes;
    for (int b : kb_order) if (classes.empty() || classes.back() != ucost[b]) classes.push_back(ucost[b]);
    std::vector<std::vector<std::pair<int64_t, int>>> assigned(P);
    for (double cls : classes) {
      for (int64_t t = 0; t < T; ++t)
        for (int kb = 0; kb < nb; ++kb) {
          if (ucost[kb] != cls) continue;
          auto [l, c] = pq.top();
          pq.pop();
          assigned[c].push_back({t, kb});
          pq.push({l + ucost[kb], c});
        }
    }
    for (int c = 0; c < P; ++c) {
      std::sort(assigned[c].begin(), assigned[c].end());
      for (auto& [t, kb] : assigned[c]) add_unit(c, t, kb);
    }
  } else {
    const int64_t full_waves = std::max<int64_t>(0, T / P - 1);
    const int64_t t_dp = full_waves * P;
    for (int64_t ti = 0; ti < t_dp; ++ti) {
      runs[ti % P].push_back({order[(size_t)ti], 0, nb});
      load[ti % P] += tile_cost;
    }
    const int64_t t_sk = T - t_dp;
    if (t_sk > 0) {
      std::vector<double> seq((size_t)(t_sk * nb));
      for (int64_t i = 0; i < t_sk; ++i)
        for (int kb = 0; kb < nb; ++kb) seq[i * nb + kb] = ucost[kb];
      std::vector<int64_t> cut = best_contiguous_cuts(seq, P);
      for (int c = 0; c < P; ++c)
        for (int64_t u = cut[c]; u < cut[c + 1]; ++u) add_unit(c, order[(size_t)(t_dp + u / nb)], (int)(u % nb));
    }
  }

  // ---- segments -> work items
  struct SegRef { int cta; size_t idx; };
  std::map<int64_t, std::vector<SegRef>> by_tile;
  for (int c = 0; c < P; ++c)
    for (size_t i = 0; i < runs[c].size(); ++i) by_tile[runs[c][i].tile].push_back({c, i});
  std::vector<std::vector<WorkItem>> per(P);
  for (int c = 0; c < P; ++c) per[c].resize(runs[c].size());
  p.n_split_tiles = 0;
  p.max_segments = 1;
  int32_t fix = 0;
  p.fix_info.clear();
  for (auto& [tile, segs] : by_tile) {
    std::sort(segs.begin(), segs.end(), [&](const SegRef& a, const SegRef& b) {
      return runs[a.cta][a.idx].kb0 < runs[b.cta][b.idx].kb0;
    });
    const int nseg = (int)segs.size();
    if (nseg > 255) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "a tile split into more than 255 segments");
    const bool split = nseg > 1;
    if (split) { p.n_split_tiles++; p.max_segments = std::max(p.max_segments, nseg); }
    for (int s = 0; s < nseg; ++s) {
      const Run& r = runs[segs[s].cta][segs[s].idx];
      WorkItem w{};
      w.tile = (int32_t)tile; w.kb_begin = r.kb0 * kgran; w.kb_end = std::min(r.kb1 * kgran, nkb);
      w.flags = (split ? 1 : 0) | (s == 0 ? 2 : 0) | (s << 8) | (nseg << 16);
      w.fix = split ? fix : -1;
      per[segs[s].cta][segs[s].idx] = w;
    }
    if (split) {
      p.fix_info.push_back((int32_t)tile);
      p.fix_info.push_back(nseg);
      ++fix;
    }
  }
  p.cta_begin.assign(P + 1, 0);
  p.items.clear();
  for (int c = 0; c < P; ++c) {
    p.cta_begin[c] = (int32_t)p.items.size();
    // non-owner segments first (they never wait), then the rest in unit order
    std::stable_partition(per[c].begin(), per[c].end(), [](const WorkItem& w) { return (w.flags & 2) == 0; });
    for (auto& w : per[c]) p.items.push_back(w);
  }
  p.cta_begin[P] = (int32_t)p.items.size();
  p.max_cost = *std::max_element(load.begin(), load.end());
  p.mean_cost = std::accumulate(load.begin(), load.end(), 0.0) / P;
  const size_t part = (size_t)p.tile_n * p.tile_w * sizeof(float);
  // partial slots: [split tile][segment] (the decode kernel stores every segment's partial and
  // the last arriver sums them; the prefill kernel uses slots 1.. for the non-owner segments);
  // flags / arrival counters after them
  const size_t n_part = (size_t)p.n_split_tiles * (size_t)p.max_segments;
  p.ws_flags_off = n_part * part;
  p.ws_bytes = p.n_split_tiles ? p.ws_flags_off + (size_t)p.n_split_tiles * p.max_segments * 2 * sizeof(uint32_t) : 0;
  p.ws_bytes = (p.ws_bytes + 255) / 256 * 256;
  if (p.ws_bytes > ((size_t)8 << 30)) return fail(COMET_ERR_UNSUPPORTED_SHAPE, "schedule needs more than 8 GiB of fix-up workspace");
  return COMET_OK;
}

}  // namespace comet
