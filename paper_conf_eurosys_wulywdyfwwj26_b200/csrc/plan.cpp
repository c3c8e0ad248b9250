// plan.cpp -- see plan.h.
#include "plan.h"

#include "common.h"

#include <algorithm>
#include <numeric>

namespace gr {

using u128 = unsigned __int128;
static constexpr uint64_t kPsPerSec = 1000000000000ull;

// Uplink groups: explicit ids win; otherwise i ~ j when their concurrent H2D
// sum is within 15% of the better solo bandwidth (shared uplink, L131); the
// groups are the connected components (union-find).
static std::vector<std::vector<int>> build_groups(const grouter_config &c) {
  const int n = (int)c.n_gpus;
  std::vector<int> parent(n);
  std::iota(parent.begin(), parent.end(), 0);
  auto find = [&](int x) {
    while (parent[x] != x) x = parent[x] = parent[parent[x]];
    return x;
  };
  auto unite = [&](int a, int b) {
    a = find(a), b = find(b);
    if (a != b) parent[std::max(a, b)] = std::min(a, b);
  };
  if (c.flags & GROUTER_NO_TOPOLOGY) {  // ablation "TA off" (R48): no shared uplinks assumed
    std::vector<std::vector<int>> g(n);
    for (int i = 0; i < n; ++i) g[i] = {i};
    return g;
  }
  bool explicit_ids = false;
  for (int i = 0; i < n; ++i) explicit_ids |= c.uplink_group[i] >= 0;
  for (int i = 0; i < n; ++i)
    for (int j = i + 1; j < n; ++j) {
      bool shared;
      if (explicit_ids) {
        shared = c.uplink_group[i] >= 0 && c.uplink_group[i] == c.uplink_group[j];
      } else {
        // either direction of the (normally symmetric) matrix may witness it
        u128 best = std::max(c.h2d_Bps[i], c.h2d_Bps[j]);
        u128 pij = std::min(c.h2d_pair_Bps[i][j], c.h2d_pair_Bps[j][i]);
        shared = (u128)100 * pij <= (u128)115 * best;
      }
      if (shared) unite(i, j);
    }
  std::vector<std::vector<int>> g;
  std::vector<int> slot(n, -1);
  for (int i = 0; i < n; ++i) {  // ascending i => groups ordered by lowest index
    int r = find(i);
    if (slot[r] < 0) {
      slot[r] = (int)g.size();
      g.emplace_back();
    }
    g[slot[r]].push_back(i);
  }
  return g;
}

void Planner::build(const grouter_config &c) {
  cfg = c;
  const int n = (int)c.n_gpus;
  groups = build_groups(c);
  routes.assign(n, {});
  paths.assign(n, {});
  const bool multipath = !(c.flags & GROUTER_NO_MULTIPATH);
  for (int d = 0; d < n; ++d) {
    auto &R = routes[d];
    R.push_back(d);                                  // d represents its own group (R10)
    if (multipath)
      for (auto &g : groups) {
        if (std::find(g.begin(), g.end(), d) != g.end()) continue;
        int r = g.front();                           // lowest index represents it (R10)
        if (c.p2p[r][d]) R.push_back(r);
      }
    uint64_t bmax = 0;
    for (int r : R) {
      PathModel p;
      p.route_gpu = r;
      p.alpha_ps = c.h2d_alpha_ps[r];
      if (r == d) {
        p.beta_Bps = c.h2d_Bps[d];
        p.phi_ps = c.h2d_phi_ps[d];
      } else {  // PCIe of r, then one NVLink hop r -> d
        p.beta_Bps = std::min(c.h2d_Bps[r], c.nvl_Bps);
        p.phi_ps = c.h2d_phi_ps[r] + c.relay_phi_ps;
      }
      if (p.beta_Bps == 0) p.beta_Bps = 1;
      bmax = std::max(bmax, p.beta_Bps);
      paths[d].push_back(p);
    }
    const uint64_t C = c.chunk_bytes, g = c.granule;
    for (auto &p : paths[d]) {  // C_p proportional to capacity (L242), >= one granule
      uint64_t cp = (uint64_t)(((u128)C * p.beta_Bps) / ((u128)bmax * g)) * g;
      p.chunk = std::max(g, cp);
    }
  }
}

// T_p(m): time for m granules on path p, in ps.
static u128 path_time(uint64_t m, const PathModel &p, uint64_t g) {
  if (m == 0) return 0;
  u128 bytes = (u128)m * g;
  u128 chunks = (bytes + p.chunk - 1) / p.chunk;
  u128 xfer = (bytes * kPsPerSec + p.beta_Bps - 1) / p.beta_Bps;
  return (u128)p.phi_ps + chunks * p.alpha_ps + xfer;
}

// Largest m <= N with T_p(m) <= T (T_p is non-decreasing in m).  The
// ceilings put T_p(m) between L(m) = phi + m*r and L(m) + alpha + 1 ps, with
// r = g*alpha/C + g*1e12/beta per granule, so the answer lies in a window of
// about (alpha + 1)/r granules around (T - phi)/r; the window is verified
// (and widened if rounding misplaced it) with the exact T_p before the
// bisection, so the result is the exact one.
static uint64_t path_cap(u128 T, uint64_t N, const PathModel &p, uint64_t g) {
  if (path_time(N, p, g) <= T) return N;
  if (T < (u128)p.phi_ps) return 0;
  const double r = (double)g * (double)p.alpha_ps / (double)p.chunk + (double)g * 1e12 / (double)p.beta_Bps;
  const double span = (double)(T - (u128)p.phi_ps);
  const double a = (span - (double)p.alpha_ps - 1.0) / r, b = span / r;
  uint64_t lo = a <= 1.0 ? 0 : (uint64_t)a - 1, hi = b >= (double)N ? N : (uint64_t)b + 1;
  if (hi > N) hi = N;
  if (lo > hi) lo = hi;
  while (lo > 0 && path_time(lo, p, g) > T) lo = lo > 64 ? lo - 64 : 0;  // lo must be feasible
  while (hi < N && path_time(hi + 1, p, g) <= T) hi = std::min<uint64_t>(N, hi + 64);  // hi+1 infeasible
  while (lo < hi) {
    uint64_t mid = lo + (hi - lo + 1) / 2;
    if (path_time(mid, p, g) <= T) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

// O6 split of n bytes over paths P (route order): exact min-makespan shares,
// canonical fill, interleaved layout with C_p-sized chunks.
void split_plan(const std::vector<PathModel> &P, uint64_t n, uint64_t g, std::vector<grouter_chunk> &out) {
  out.clear();
  if (n == 0 || P.empty()) return;
  const uint64_t N = ceil_div(n, g);
  if (P.size() == 1) {  // one path carries every granule: chunks of C_p
    for (uint64_t off = 0; off < n; off += P[0].chunk)
      out.push_back({off, std::min<uint64_t>(P[0].chunk, n - off), 0, (int32_t)P[0].route_gpu});
    return;
  }
  // 1. T* = min { T : sum_p cap_p(T) >= N }  (bisection on integer ps)
  u128 lo = 0, hi = path_time(N, P[0], g);
  while (lo < hi) {
    u128 mid = lo + (hi - lo) / 2;
    u128 tot = 0;
    for (auto &p : P) tot += path_cap(mid, N, p, g);
    if (tot >= N) hi = mid;
    else lo = mid + 1;
  }
  // 2. canonical shares: fill paths in route order up to cap_p(T*)
  std::vector<uint64_t> rem(P.size());
  uint64_t left = N;
  for (size_t i = 0; i < P.size(); ++i) {
    rem[i] = std::min(path_cap(lo, N, P[i], g), left);
    left -= rem[i];
  }
  // 3. interleaved rounds: each path emits up to C_p/g granules per round
  uint64_t off = 0;
  bool any = true;
  while (any) {
    any = false;
    for (size_t i = 0; i < P.size(); ++i) {
      if (!rem[i]) continue;
      uint64_t m = std::min(P[i].chunk / g, rem[i]);
      out.push_back({off, m * g, (int32_t)i, (int32_t)P[i].route_gpu});
      off += m * g;
      rem[i] -= m;
      any = true;
    }
  }
  out.back().bytes = n - out.back().offset;  // clip the final chunk to n
}

// C_p = max(g, floor(C * beta_p / beta_max / g) * g)  (L242, R2)
void size_chunks(std::vector<PathModel> &P, uint64_t C, uint64_t g) {
  uint64_t bmax = 0;
  for (auto &p : P) bmax = std::max(bmax, p.beta_Bps);
  for (auto &p : P) {
    uint64_t cp = (uint64_t)(((u128)C * p.beta_Bps) / ((u128)bmax * g)) * g;
    p.chunk = std::max(g, cp);
  }
}

void Planner::plan_h2d(int d, uint64_t n, std::vector<grouter_chunk> &out) const {
  std::lock_guard<std::mutex> lk(cache_mu);
  auto &m = cache[d];
  auto it = m.find(n);
  if (it != m.end()) {
    out = it->second;
    return;
  }
  split_plan(paths[d], n, cfg.granule, out);
  if (m.size() >= 256) m.clear();  // bounded; sizes in a workload repeat
  m.emplace(n, out);
}

void Planner::plan_single(uint64_t n, int route_gpu, std::vector<grouter_chunk> &out) const {
  out.clear();
  for (uint64_t o = 0; o < n; o += cfg.chunk_bytes)
    out.push_back({o, std::min<uint64_t>(cfg.chunk_bytes, n - o), 0, route_gpu});
}

void Planner::plan(int src, int dst, uint64_t n, std::vector<grouter_chunk> &out, bool pool_src) const {
  out.clear();
  if (n == 0 || (src == GROUTER_HOST && dst == GROUTER_HOST)) return;
  if (src == GROUTER_HOST) plan_h2d(dst, n, out);
  // gFn-host (L178, Fig. 5a): GPU src -> route GPUs -> host.  PCIe is
  // calibrated in the host->GPU direction and taken as symmetric, so the
  // split over R(src) is the host->GPU plan of src (R45)
  else if (dst == GROUTER_HOST && pool_src && (cfg.flags & GROUTER_D2H_MULTIPATH)) plan_h2d(src, n, out);
  else plan_single(n, src, out);  // D2D / same-GPU copy / D2H: source GPU's engine
}

}  // namespace gr
