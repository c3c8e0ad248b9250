// stride.h -- tenant share scheduler of one server (one shared link/engine).
//
// PAPER.md L193 (chunks of each function are scheduled proportionally to
// their allocated bandwidth), L229 (batches of 5 chunks; new functions join
// at the next batch, which bounds the preemption delay).  Stride scheduling
// (readings R6, R9): a batch is <= batch_chunks chunks of ONE tenant; the
// backlogged tenant with minimum pass goes next (ties -> lower id); its pass
// advances by ceil(bytes * 2^20 / weight); a tenant that becomes backlogged
// joins at max(pass, V), V = pass of the last dispatched tenant.
#pragma once

#include <cstdint>
#include <deque>
#include <map>
#include <vector>

namespace gr {

template <class Item>
struct Stride {
  struct Tenant {
    std::deque<Item> q;
    uint64_t pass = 0;
  };
  uint32_t batch = 5;
  uint64_t V = 0;
  std::map<uint32_t, Tenant> tenants;  // ordered by id: ties resolve to the lower id
  uint64_t backlog_items = 0;

  // bytes(item) must be provided by Item::bytes
  void enqueue(uint32_t t, const Item &it) {
    Tenant &tn = tenants[t];
    if (tn.q.empty()) tn.pass = tn.pass > V ? tn.pass : V;  // join rule
    tn.q.push_back(it);
    ++backlog_items;
  }
  bool empty() const { return backlog_items == 0; }

  // Forgets idle tenants whose pass is <= V: a tenant that re-joins later gets
  // max(pass, V) = V either way, so this changes no dispatch decision; it
  // bounds the table when workflows are short-lived (one id per request).
  void prune() {
    for (auto it = tenants.begin(); it != tenants.end();)
      if (it->second.q.empty() && it->second.pass <= V) it = tenants.erase(it);
      else ++it;
  }

  // The pass/V updates dispatch() makes when tenant t, alone on an idle
  // server, has n bytes in chunks of `chunk` bytes (all full but the last)
  // dispatched in batches -- for transfers that bypass the queues (a direct
  // launch on an idle SM-copy server), so later contention sees the same
  // passes as if the chunks had been queued.
  void account_solo(uint32_t t, uint64_t n, uint64_t chunk, uint64_t w) {
    Tenant &tn = tenants[t];
    if (tn.q.empty()) tn.pass = tn.pass > V ? tn.pass : V;  // join rule
    if (w == 0) w = 1;
    const uint64_t per_batch = chunk * batch;
    while (n) {
      const uint64_t bytes = n < per_batch ? n : per_batch;
      V = tn.pass;
      unsigned __int128 s = ((unsigned __int128)bytes << 20);
      tn.pass += (uint64_t)((s + w - 1) / w);
      n -= bytes;
    }
  }

  // Pops the next batch into `out`; returns the tenant id, or UINT32_MAX if idle.
  template <class WeightFn>
  uint32_t dispatch(WeightFn weight_of, std::vector<Item> &out, uint64_t *bytes_out = nullptr,
                    uint64_t *pass_after = nullptr) {
    out.clear();
    uint32_t best = UINT32_MAX;
    uint64_t best_pass = 0;
    for (auto &kv : tenants) {
      if (kv.second.q.empty()) continue;
      if (best == UINT32_MAX || kv.second.pass < best_pass) {
        best = kv.first;
        best_pass = kv.second.pass;
      }
    }
    if (best == UINT32_MAX) return best;
    Tenant &tn = tenants[best];
    uint64_t bytes = 0;
    while (!tn.q.empty() && out.size() < batch) {
      bytes += tn.q.front().bytes;
      out.push_back(tn.q.front());
      tn.q.pop_front();
      --backlog_items;
    }
    uint64_t w = weight_of(best);
    if (w == 0) w = 1;
    V = tn.pass;
    unsigned __int128 s = ((unsigned __int128)bytes << 20);
    tn.pass += (uint64_t)((s + w - 1) / w);
    if (bytes_out) *bytes_out = bytes;
    if (pass_after) *pass_after = tn.pass;
    return best;
  }
};

}  // namespace gr
