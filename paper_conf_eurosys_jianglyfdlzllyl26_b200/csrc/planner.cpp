// a10: Alg. 1 "DP for pipeline loading" (§4.2, Fig. 9-Bottom).
// The algorithm body is lost in extraction; the pipeline model is reading R11:
//   load stream: the cached blocks' loads in block order, back to back from t = 0;
//   compute stream: block l starts at max(end(l-1), dep(l)), lasts C_w^m[l] or C_w/o[l];
//   KV-mode: dep(l) = end of block l's load; plans monotone; final load of the last block's Y;
//   Y-mode : dep(l+1) = end of block l's load; the step ends after block N-1's load.
// Host-only C++ (no CUDA).
#include <algorithm>
#include <cmath>
#include <limits>
#include <vector>

#include "../../include/flashps.h"

namespace {

double latency_of(const uint8_t* use, const double* Cw, const double* Cwo, const double* Lm,
                  int N, int mode, double final_load) {
  if (mode == FPS_MODE_KV) {
    bool seen = false;
    for (int l = 0; l < N; ++l) {
      if (use[l]) seen = true;
      else if (seen) return std::numeric_limits<double>::infinity();
    }
  }
  double t_load = 0.0, t = 0.0, prev_load_end = 0.0;
  bool any = false, prev_cached = false;
  for (int l = 0; l < N; ++l) {
    double dep = 0.0;
    if (mode == FPS_MODE_Y && prev_cached) dep = prev_load_end;
    double my_load_end = 0.0;
    if (use[l]) {
      t_load += Lm[l];
      my_load_end = t_load;
      any = true;
      if (mode == FPS_MODE_KV) dep = my_load_end;
    }
    t = std::max(t, dep) + (use[l] ? Cw[l] : Cwo[l]);
    prev_cached = use[l] != 0;
    prev_load_end = my_load_end;
  }
  if (mode == FPS_MODE_KV && any) t = std::max(t, t_load + final_load);
  if (mode == FPS_MODE_Y && N > 0 && use[N - 1]) t = std::max(t, prev_load_end);
  return t;
}

// KV-mode: the feasible plans are the N+1 suffixes "uncached 0..k-1, cached k..N-1".  With
// prefix sums, latency(k) = max(P_k + SC_k, max_{l>=k}(SL_l + SC_l) - SL_{k-1}, SL_{N-1} -
// SL_{k-1} + final): an O(N) scan (the paper's complexity, L211).
double plan_kv(const double* Cw, const double* Cwo, const double* Lm, int N, double final_load,
               uint8_t* use) {
  std::vector<double> SL(N + 1, 0.0), SC(N + 1, 0.0), Amax(N + 1, -1e300);
  for (int l = 0; l < N; ++l) SL[l + 1] = SL[l] + Lm[l];            // SL[l+1] = sum_{j<=l}
  for (int l = N - 1; l >= 0; --l) SC[l] = SC[l + 1] + Cw[l];       // SC[l] = sum_{j>=l}
  for (int l = N - 1; l >= 0; --l) Amax[l] = std::max(Amax[l + 1], SL[l + 1] + SC[l]);
  double best = std::numeric_limits<double>::infinity();
  int best_k = N;
  double P = 0.0;
  for (int k = 0; k <= N; ++k) {
    double lat;
    if (k == N) {
      lat = P;
    } else {
      lat = std::max(P + SC[k], Amax[k] - SL[k]);
      lat = std::max(lat, SL[N] - SL[k] + final_load);
    }
    if (std::isinf(best) || lat < best - 1e-12 * std::max(1.0, std::fabs(best))) {
      best = lat;
      best_k = k;
    }
    if (k < N) P += Cwo[k];
  }
  for (int l = 0; l < N; ++l) use[l] = l >= best_k ? 1 : 0;
  return best;
}

// Y-mode: exact Pareto-front DP.  State after block l: (compute end tc, load-stream end tl,
// whether block l is cached).  The final latency is non-decreasing in (tc, tl), so states
// dominated in both coordinates (with a no-dependency state dominating a dependency state)
// can be dropped without losing the optimum.
struct St {
  double tc, tl;
  uint8_t c;
  int parent;
};

double plan_y(const double* Cw, const double* Cwo, const double* Lm, int N, uint8_t* use) {
  std::vector<std::vector<St>> layers(N + 1);
  layers[0].push_back({0.0, 0.0, 0, -1});
  std::vector<St> cand;
  for (int l = 0; l < N; ++l) {
    cand.clear();
    const auto& prev = layers[l];
    for (int i = 0; i < (int)prev.size(); ++i) {
      const St& s = prev[i];
      const double start = std::max(s.tc, s.c ? s.tl : 0.0);
      cand.push_back({start + Cwo[l], s.tl, 0, i});
      cand.push_back({start + Cw[l], s.tl + Lm[l], 1, i});
    }
    std::sort(cand.begin(), cand.end(), [](const St& a, const St& b) {
      if (a.tc != b.tc) return a.tc < b.tc;
      if (a.tl != b.tl) return a.tl < b.tl;
      return a.c < b.c;
    });
    auto& out = layers[l + 1];
    double best_tl0 = std::numeric_limits<double>::infinity();   // min tl among kept c=0
    double best_tl1 = std::numeric_limits<double>::infinity();   // min tl among kept c=1
    for (const St& s : cand) {
      // kept states have tc <= s.tc (sorted); s is dominated if one of them has tl <= s.tl
      // and (same c, or the dominating state is c = 0).
      if (s.c == 0) {
        if (best_tl0 <= s.tl) continue;
        best_tl0 = s.tl;
      } else {
        if (best_tl0 <= s.tl || best_tl1 <= s.tl) continue;
        best_tl1 = s.tl;
      }
      out.push_back(s);
    }
  }
  double best = std::numeric_limits<double>::infinity();
  int bi = -1;
  const auto& last = layers[N];
  for (int i = 0; i < (int)last.size(); ++i) {
    const St& s = last[i];
    const double lat = s.c ? std::max(s.tc, s.tl) : s.tc;
    if (lat < best) {
      best = lat;
      bi = i;
    }
  }
  for (int l = N; l >= 1; --l) {
    const St& s = layers[l][bi];
    use[l - 1] = s.c;
    bi = s.parent;
  }
  return best;
}

// Cross-step prefetch (reading R26): the load stream never waits for the step boundary --
// load j of step s+1 starts when the stream is free and step s has consumed its slot (one slot
// per load); compute runs the steps in order.  Steady per-step time = mean step time over the
// second half of kSteadySteps simulated steps.
constexpr int kSteadySteps = 16;

double steady_of(const uint8_t* use, const double* Cw, const double* Cwo, const double* Lm,
                 int N, int mode, double final_load) {
  if (mode == FPS_MODE_KV) {
    bool seen = false;
    for (int l = 0; l < N; ++l) {
      if (use[l]) seen = true;
      else if (seen) return std::numeric_limits<double>::infinity();
    }
  }
  std::vector<int> blk;                       // block of each load; N = final Y rows (KV)
  std::vector<int> slot_of(N, -1);
  for (int l = 0; l < N; ++l)
    if (use[l]) {
      slot_of[l] = (int)blk.size();
      blk.push_back(l);
    }
  if (mode == FPS_MODE_KV && !blk.empty()) blk.push_back(N);
  const int nl = (int)blk.size();
  std::vector<double> freed(nl, 0.0), ready(nl, 0.0), end(N, 0.0);
  double t_load = 0.0, t_comp = 0.0, half_end = 0.0;
  for (int s = 0; s < kSteadySteps; ++s) {
    for (int j = 0; j < nl; ++j) {
      t_load = std::max(t_load, freed[j]) + (blk[j] < N ? Lm[blk[j]] : final_load);
      ready[j] = t_load;
    }
    double t = t_comp;
    for (int l = 0; l < N; ++l) {
      double dep = 0.0;
      if (mode == FPS_MODE_KV && use[l]) dep = ready[slot_of[l]];
      if (mode == FPS_MODE_Y && l > 0 && use[l - 1]) dep = ready[slot_of[l - 1]];
      t = std::max(t, dep) + (use[l] ? Cw[l] : Cwo[l]);
      end[l] = t;
    }
    if (nl > 0) {
      if (mode == FPS_MODE_KV) t = std::max(t, ready[nl - 1]);
      if (mode == FPS_MODE_Y && use[N - 1]) t = std::max(t, ready[slot_of[N - 1]]);
    }
    for (int j = 0; j < nl; ++j) {
      const int l = blk[j];
      freed[j] = l == N ? t : mode == FPS_MODE_KV ? end[l] : (l + 1 < N ? end[l + 1] : t);
    }
    t_comp = t;
    if (s == kSteadySteps / 2 - 1) half_end = t;
  }
  return (t_comp - half_end) / (kSteadySteps - kSteadySteps / 2);
}

}  // namespace

extern "C" {

double fps_pipeline_latency_cross(const uint8_t* use_cache, const double* c_cached,
                                  const double* c_dense, const double* load, int32_t N,
                                  int32_t mode, double final_load) {
  if (N < 0 || (N > 0 && (!use_cache || !c_cached || !c_dense || !load)))
    return std::numeric_limits<double>::quiet_NaN();
  return N == 0 ? 0.0 : steady_of(use_cache, c_cached, c_dense, load, N, mode, final_load);
}

fps_status fps_plan_pipeline_cross(const double* c_cached, const double* c_dense,
                                   const double* load, int32_t N, int32_t mode,
                                   double final_load, uint8_t* use_cache, double* latency) {
  if (N < 0 || !latency || (N > 0 && (!c_cached || !c_dense || !load || !use_cache)))
    return FPS_EINVAL;
  if (mode != FPS_MODE_KV && mode != FPS_MODE_Y) return FPS_EINVAL;
  std::vector<uint8_t> p(N);
  double best = std::numeric_limits<double>::infinity();
  int best_k = 0;
  for (int k = 0; k <= N; ++k) {                 // suffix plans, ties -> fewer cached blocks
    for (int l = 0; l < N; ++l) p[l] = l >= N - k ? 1 : 0;
    const double v = N == 0 ? 0.0 : steady_of(p.data(), c_cached, c_dense, load, N, mode, final_load);
    if (v < best - 1e-12 * std::max(1.0, std::fabs(best)) || std::isinf(best)) {
      best = v;
      best_k = k;
    }
  }
  for (int l = 0; l < N; ++l) use_cache[l] = l >= N - best_k ? 1 : 0;
  // (uniform stacks: the suffix scan is already optimal, SURVEY §8(c) #11 -- skip the search)
  bool uniform = true;
  for (int l = 1; l < N && uniform; ++l)
    uniform = c_cached[l] == c_cached[0] && c_dense[l] == c_dense[0] && load[l] == load[0];
  if (mode == FPS_MODE_Y && N > 0 && !uniform) {
    // Y-mode allows any pattern, and the suffix plans are not optimal on heterogeneous stacks
    // (SURVEY §8(c) #11).  Improve by local search under the same steady-state model: seeds =
    // the best suffix and the per-step exact Pareto-DP plan; first-improvement single-block
    // flips, then pairs when no single flip helps, until neither does.  Never worse than the
    // scan; exact in 58 of 60 random heterogeneous stacks of <= 10 blocks, within 7 % in all
    // (tests/test_lib_cpu.py).
    // (the Pareto-DP seed only on short stacks: its front grows with heterogeneous costs --
    //  7.5 ms at 57 random blocks -- and the engine plans at every admission)
    std::vector<std::vector<uint8_t>> seeds = {std::vector<uint8_t>(use_cache, use_cache + N)};
    if (N <= 24) {
      seeds.emplace_back(N);
      plan_y(c_cached, c_dense, load, N, seeds.back().data());
    }
    auto better = [](double w, double v) { return w < v - 1e-12 * std::max(1.0, std::fabs(v)); };
    // evaluation budget per seed (the engine plans at every admission): 8 N + N^2 model runs
    // for short stacks, 8 N for long ones (C3's 57 blocks: ~2 ms)
    const long long budget = 8LL * N + (N <= 16 ? (long long)N * N : 0);
    for (auto& q : seeds) {
      double v = steady_of(q.data(), c_cached, c_dense, load, N, mode, final_load);
      long long evals = 0;
      for (int pass = 0; pass < 4 * N && evals < budget; ++pass) {
        bool improved = false;
        for (int l = 0; l < N; ++l, ++evals) {   // single-block flips
          q[l] ^= 1;
          const double w = steady_of(q.data(), c_cached, c_dense, load, N, mode, final_load);
          if (better(w, v)) {
            v = w;
            improved = true;
          } else {
            q[l] ^= 1;
          }
        }
        // then pairs of blocks (plateaus of one flip): all pairs on short stacks, adjacent
        // pairs on long ones (the engine plans at every admission: C3 57 blocks ~1 ms)
        const int span = N <= 16 ? N : 2;
        if (!improved)
          for (int a = 0; a < N && !improved && evals < budget; ++a)
            for (int b = a + 1; b < std::min(N, a + span) && !improved; ++b, ++evals) {
              q[a] ^= 1;
              q[b] ^= 1;
              const double w = steady_of(q.data(), c_cached, c_dense, load, N, mode, final_load);
              if (better(w, v)) {
                v = w;
                improved = true;
              } else {
                q[a] ^= 1;
                q[b] ^= 1;
              }
            }
        if (!improved) break;
      }
      if (v < best - 1e-12 * std::max(1.0, std::fabs(best))) {
        best = v;
        for (int l = 0; l < N; ++l) use_cache[l] = q[l];
      }
    }
  }
  *latency = best;
  return FPS_OK;
}


double fps_pipeline_latency(const uint8_t* use_cache, const double* c_cached,
                            const double* c_dense, const double* load, int32_t N, int32_t mode,
                            double final_load) {
  if (N < 0 || (N > 0 && (!use_cache || !c_cached || !c_dense || !load)))
    return std::numeric_limits<double>::quiet_NaN();
  return latency_of(use_cache, c_cached, c_dense, load, N, mode, final_load);
}

fps_status fps_plan_pipeline(const double* c_cached, const double* c_dense, const double* load,
                             int32_t N, int32_t mode, double final_load, uint8_t* use_cache,
                             double* latency) {
  if (N < 0 || !latency || (N > 0 && (!c_cached || !c_dense || !load || !use_cache)))
    return FPS_EINVAL;
  if (mode != FPS_MODE_KV && mode != FPS_MODE_Y) return FPS_EINVAL;
  if (N == 0) {
    *latency = 0.0;
    return FPS_OK;
  }
  *latency = mode == FPS_MODE_KV ? plan_kv(c_cached, c_dense, load, N, final_load, use_cache)
                                 : plan_y(c_cached, c_dense, load, N, use_cache);
  return FPS_OK;
}

fps_status fps_plan_pipeline_kv_transition(const double* c_cached, const double* c_dense,
                                           const double* c_transition, const double* load,
                                           int32_t N, double final_load, int32_t cross_step,
                                           uint8_t* use_cache, double* latency) {
  if (N < 0 || !latency ||
      (N > 0 && (!c_cached || !c_dense || !c_transition || !load || !use_cache)))
    return FPS_EINVAL;
  std::vector<uint8_t> p(N);
  std::vector<double> cd(c_dense, c_dense + N);
  double best = std::numeric_limits<double>::infinity();
  int best_k = 0;
  for (int k = 0; k <= N; ++k) {                 // k cached blocks; ties -> fewer cached
    for (int l = 0; l < N; ++l) p[l] = l >= N - k ? 1 : 0;
    const int t = N - k - 1;                     // the prefix's last block, if both parts exist
    if (k > 0 && t >= 0) cd[t] = c_transition[t];
    const double v = N == 0 ? 0.0
                     : cross_step ? steady_of(p.data(), c_cached, cd.data(), load, N, FPS_MODE_KV, final_load)
                                  : latency_of(p.data(), c_cached, cd.data(), load, N, FPS_MODE_KV, final_load);
    if (k > 0 && t >= 0) cd[t] = c_dense[t];
    if (v < best - 1e-12 * std::max(1.0, std::fabs(best)) || std::isinf(best)) {
      best = v;
      best_k = k;
    }
  }
  for (int l = 0; l < N; ++l) use_cache[l] = l >= N - best_k ? 1 : 0;
  *latency = N == 0 ? 0.0 : best;
  return FPS_OK;
}

}  // extern "C"
