// paths.cpp -- contention-aware NVLink path selection, Algorithm 1 in full
// (§4.3.3; readings R11, R46 in DESIGN.md).
//
// Host-side planner state: the topology matrix Topo (GPU and switch nodes,
// directed B/s), the real-time free-bandwidth matrix BW and the active
// allocations (function, path, b).  select() runs Alg. 1 for one function:
// direct priority (L235), free shortest paths (lines 1-7, b_min update L237),
// then busy paths with bandwidth balancing while the endpoints are
// unsaturated (lines 8-14, L237); functions moved off a path re-run the free
// phase.  On an NVSwitch node (HGX B200) every pair gets only its direct
// path; the data path's D2D copies therefore use the direct route, and this
// planner serves asymmetric meshes (DGX-V100 style) and the NVLink chunk plan
// of L242.
#include <algorithm>
#include <cstring>
#include <new>
#include <vector>

#include "../../include/grouter.h"
#include "common.h"
#include "plan.h"

namespace gr {
namespace {

using Path = std::vector<int>;

struct Alloc {
  uint32_t func;
  Path path;
  uint64_t b;
};

}  // namespace
}  // namespace gr

struct grouter_paths {
  int n = 0, n_gpus = 0, H = 3;
  std::vector<uint64_t> topo, bw;  // n x n, row = from
  std::vector<gr::Alloc> alloc;     // allocation order

  uint64_t &B(int u, int v) { return bw[(size_t)u * n + v]; }
  uint64_t T(int u, int v) const { return topo[(size_t)u * n + v]; }

  std::vector<gr::Path> candidates(int gs, int gd) const {
    std::vector<gr::Path> out;
    if (gs == gd) return out;
    gr::Path p{gs};
    std::vector<char> on(n, 0);
    on[gs] = 1;
    // depth-first, neighbours ascending; sorted by (edge count, sequence) after
    struct Rec {
      const grouter_paths *t;
      int gd;
      std::vector<gr::Path> *out;
      gr::Path *p;
      std::vector<char> *on;
      void go() {
        int u = p->back();
        if (u == gd) {
          out->push_back(*p);
          return;
        }
        if ((int)p->size() - 1 == t->H) return;
        for (int v = 0; v < t->n; ++v)
          if (t->T(u, v) > 0 && !(*on)[v]) {
            (*on)[v] = 1;
            p->push_back(v);
            go();
            p->pop_back();
            (*on)[v] = 0;
          }
      }
    } rec{this, gd, &out, &p, &on};
    rec.go();
    std::stable_sort(out.begin(), out.end(), [](const gr::Path &a, const gr::Path &b) {
      if (a.size() != b.size()) return a.size() < b.size();
      return a < b;
    });
    return out;
  }

  static bool has_edge(const gr::Path &p, int u, int v) {
    for (size_t i = 0; i + 1 < p.size(); ++i)
      if (p[i] == u && p[i + 1] == v) return true;
    return false;
  }
  static bool share_edge(const gr::Path &a, const gr::Path &b) {
    for (size_t i = 0; i + 1 < a.size(); ++i)
      if (has_edge(b, a[i], a[i + 1])) return true;
    return false;
  }
  uint64_t bw_out(int g) {
    uint64_t s = 0;
    for (int v = 0; v < n; ++v) s += B(g, v);
    return s;
  }
  uint64_t bw_in(int g) {
    uint64_t s = 0;
    for (int u = 0; u < n; ++u) s += B(u, g);
    return s;
  }
  bool saturated(int gs, int gd) { return bw_out(gs) == 0 || bw_in(gd) == 0; }
  uint64_t bmin(const gr::Path &p) {
    uint64_t m = UINT64_MAX;
    for (size_t i = 0; i + 1 < p.size(); ++i) m = std::min(m, B(p[i], p[i + 1]));
    return m;
  }
  bool idle(const gr::Path &p) {
    for (size_t i = 0; i + 1 < p.size(); ++i)
      if (B(p[i], p[i + 1]) != T(p[i], p[i + 1])) return false;
    return true;
  }
  void take(uint32_t f, const gr::Path &p) {
    const uint64_t b = bmin(p);
    for (size_t i = 0; i + 1 < p.size(); ++i) B(p[i], p[i + 1]) -= b;
    alloc.push_back({f, p, b});
  }
  void drop(size_t k) {
    const gr::Alloc &a = alloc[k];
    for (size_t i = 0; i + 1 < a.path.size(); ++i) B(a.path[i], a.path[i + 1]) += a.b;
    alloc.erase(alloc.begin() + (long)k);
  }
  uint64_t total(uint32_t f) const {
    uint64_t s = 0;
    for (auto &a : alloc)
      if (a.func == f) s += a.b;
    return s;
  }
  size_t npaths(uint32_t f) const {
    size_t c = 0;
    for (auto &a : alloc) c += a.func == f;
    return c;
  }
  void free_phase(uint32_t f, int gs, int gd, const std::vector<gr::Path> &cands) {
    for (auto &p : cands) {
      if (saturated(gs, gd)) return;
      if (idle(p)) take(f, p);
    }
  }

  struct Moved {
    uint32_t func;
    int gs, gd;
  };

  void select(uint32_t f, int gs, int gd) {
    const auto cands = candidates(gs, gd);
    std::vector<Moved> moved;
    // direct priority (L235): other functions' indirect routes give the direct edge back
    if (T(gs, gd) > 0)
      for (size_t k = 0; k < alloc.size();) {
        const gr::Alloc &a = alloc[k];
        if (a.func != f && a.path.size() > 2 && has_edge(a.path, gs, gd)) {
          moved.push_back({a.func, a.path.front(), a.path.back()});
          drop(k);
        } else {
          ++k;
        }
      }
    free_phase(f, gs, gd, cands);  // lines 1-7
    if (!saturated(gs, gd)) {      // lines 8-14
      for (auto &p : cands) {
        if (saturated(gs, gd)) break;
        bool mine = false;
        for (auto &a : alloc)
          if (a.func == f && share_edge(a.path, p)) mine = true;
        if (mine) continue;
        if (bmin(p) > 0) {  // busy but not full: share what is left
          take(f, p);
          continue;
        }
        std::vector<size_t> holders;
        for (size_t k = 0; k < alloc.size(); ++k)
          if (alloc[k].func != f && share_edge(alloc[k].path, p)) holders.push_back(k);
        if (holders.empty()) continue;
        bool ok = true;
        for (size_t k : holders) {
          const uint32_t h = alloc[k].func;
          size_t mine_h = 0;
          for (size_t j : holders) mine_h += alloc[j].func == h;
          if (!(total(h) > total(f) && npaths(h) > mine_h)) ok = false;
        }
        if (!ok) continue;
        // bandwidth_balancing: the holders give the path up (highest index first
        // keeps the remaining indices valid; moved keeps allocation order)
        std::vector<Moved> mv;
        for (size_t k : holders) mv.push_back({alloc[k].func, alloc[k].path.front(), alloc[k].path.back()});
        for (size_t i = holders.size(); i-- > 0;) drop(holders[i]);
        moved.insert(moved.end(), mv.begin(), mv.end());
        if (bmin(p) > 0) take(f, p);
      }
    }
    for (auto &m : moved) free_phase(m.func, m.gs, m.gd, candidates(m.gs, m.gd));
  }

  void release(uint32_t f) {
    for (size_t k = 0; k < alloc.size();) {
      if (alloc[k].func == f) drop(k);
      else ++k;
    }
  }
};

namespace {
void fill_path(const gr::Alloc &a, grouter_path &o) {
  std::memset(&o, 0, sizeof(o));
  o.bw_Bps = a.b;
  o.func = a.func;
  o.n_nodes = (uint32_t)a.path.size();
  for (size_t i = 0; i < a.path.size() && i < GROUTER_MAX_PATH_NODES; ++i) o.nodes[i] = a.path[i];
}
}  // namespace

extern "C" {

grouter_paths *grouter_paths_new(uint32_t n_nodes, uint32_t n_gpus, const uint64_t *topo, uint32_t max_edges) {
  if (!topo || n_nodes == 0 || n_nodes > GROUTER_MAX_PATH_GRAPH || n_gpus > n_nodes || max_edges == 0 ||
      max_edges + 1 > GROUTER_MAX_PATH_NODES)
    return nullptr;
  auto *t = new (std::nothrow) grouter_paths();
  if (!t) return nullptr;
  t->n = (int)n_nodes;
  t->n_gpus = (int)n_gpus;
  t->H = (int)max_edges;
  t->topo.assign(topo, topo + (size_t)n_nodes * n_nodes);
  for (uint32_t i = 0; i < n_nodes; ++i) t->topo[(size_t)i * n_nodes + i] = 0;  // no self loops
  t->bw = t->topo;
  return t;
}

void grouter_paths_free(grouter_paths *t) { delete t; }

grouter_status grouter_paths_select(grouter_paths *t, uint32_t func, int32_t gs, int32_t gd, grouter_path *out,
                                    uint32_t cap, uint32_t *n_out) {
  if (!t || !n_out || gs < 0 || gd < 0 || gs >= t->n_gpus || gd >= t->n_gpus || gs == gd)
    return GROUTER_EINVAL;
  for (auto &a : t->alloc)
    if (a.func == func) return GROUTER_ESTATE;  // one selection per function until release
  t->select(func, gs, gd);
  uint32_t k = 0;
  for (auto &a : t->alloc)
    if (a.func == func) {
      if (out && k < cap) fill_path(a, out[k]);
      ++k;
    }
  *n_out = k;
  return k > cap ? GROUTER_EINVAL : GROUTER_OK;
}

grouter_status grouter_paths_release(grouter_paths *t, uint32_t func) {
  if (!t) return GROUTER_EINVAL;
  t->release(func);
  return GROUTER_OK;
}

grouter_status grouter_paths_table(grouter_paths *t, grouter_path *out, uint32_t cap, uint32_t *n_out) {
  if (!t || !n_out) return GROUTER_EINVAL;
  *n_out = (uint32_t)t->alloc.size();
  if (t->alloc.size() > cap || (!out && !t->alloc.empty())) return GROUTER_EINVAL;
  for (size_t i = 0; i < t->alloc.size(); ++i) fill_path(t->alloc[i], out[i]);
  return GROUTER_OK;
}

grouter_status grouter_paths_plan(grouter_paths *t, uint32_t func, uint64_t n, uint64_t chunk_bytes,
                                  uint64_t granule, uint64_t relay_phi_ps, grouter_chunk *out, uint64_t cap,
                                  uint64_t *n_out) {
  if (!t || !n_out || chunk_bytes == 0 || granule == 0) return GROUTER_EINVAL;
  std::vector<gr::PathModel> P;
  for (auto &a : t->alloc)
    if (a.func == func) {
      gr::PathModel m{};
      int relays = 0, first = -1;
      for (size_t i = 1; i + 1 < a.path.size(); ++i)
        if (a.path[i] < t->n_gpus) {
          if (first < 0) first = a.path[i];
          ++relays;
        }
      m.route_gpu = first >= 0 ? first : a.path.front();
      m.alpha_ps = 0;
      m.beta_Bps = a.b;
      m.phi_ps = (uint64_t)relays * relay_phi_ps;
      P.push_back(m);
    }
  std::vector<grouter_chunk> plan;
  if (!P.empty()) {
    gr::size_chunks(P, chunk_bytes, granule);
    gr::split_plan(P, n, granule, plan);
  }
  *n_out = plan.size();
  if (plan.size() > cap || (!out && !plan.empty())) return GROUTER_EINVAL;
  std::copy(plan.begin(), plan.end(), out);
  return GROUTER_OK;
}

}  // extern "C"
