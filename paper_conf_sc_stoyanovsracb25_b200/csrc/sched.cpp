// sched.cpp — the task manager of the paper's control plane, native and host-only (NEXT-1).
//
// PAPER.md §3.3-3.5 and §6:
//  * swap-in requests become memory reservations kept in a priority queue; several are granted at
//    once when memory suffices;
//  * if memory is short, victims are chosen among the running backends by the demand-aware policy:
//    shorter request queue first, then oldest last-accessed time;
//  * victims are evicted one at a time, re-checking free memory after each, and a backend being
//    evicted is write-locked;
//  * each backend's GPU topology is fixed at init and its per-GPU reservations are acquired and
//    released together.
// Readings where the paper is silent are DESIGN.md §3 readings 20-23 (shared with oracle/policy.py,
// which implements the same definition independently in plain Python).
#include <algorithm>
#include <cstring>
#include <map>
#include <set>
#include <tuple>
#include <vector>

#include "../../include/swap.h"

namespace {

struct Backend {
  std::vector<uint64_t> need;
  bool resident = false;
  bool locked = false;
  uint32_t queue = 0;
  double last_access = 0.0;
};

}  // namespace

struct swap_sched {
  std::vector<uint64_t> capacity;
  std::map<uint32_t, Backend> backends;
  std::set<std::tuple<double, uint64_t, uint32_t>> pending;  // (priority, arrival seq, backend)
  uint64_t seq = 0;

  uint64_t used(size_t g) const {
    uint64_t u = 0;
    for (const auto& kv : backends)
      if (kv.second.resident) u += kv.second.need[g];
    return u;
  }

  // Victims in eviction order; false if infeasible.
  bool plan(uint32_t id, std::vector<uint32_t>* victims) const {
    victims->clear();
    const Backend& req = backends.at(id);
    if (req.resident) return true;
    const size_t G = capacity.size();
    std::vector<int64_t> free(G);
    for (size_t g = 0; g < G; ++g) free[g] = (int64_t)capacity[g] - (int64_t)used(g);
    for (;;) {
      std::vector<size_t> short_gpus;
      for (size_t g = 0; g < G; ++g)
        if (req.need[g] > 0 && free[g] < (int64_t)req.need[g]) short_gpus.push_back(g);
      if (short_gpus.empty()) return true;
      const Backend* best = nullptr;
      uint32_t best_id = 0;
      for (const auto& kv : backends) {
        const Backend& b = kv.second;
        if (!b.resident || b.locked || kv.first == id) continue;
        if (std::find(victims->begin(), victims->end(), kv.first) != victims->end()) continue;
        bool helps = false;
        for (size_t g : short_gpus) helps |= b.need[g] > 0;
        if (!helps) continue;
        // tier 1: shorter queue; tier 2: older last access; then lower id (map order)
        if (!best || b.queue < best->queue || (b.queue == best->queue && b.last_access < best->last_access)) {
          best = &b;
          best_id = kv.first;
        }
      }
      if (!best) return false;
      victims->push_back(best_id);
      for (size_t g = 0; g < G; ++g) free[g] += (int64_t)best->need[g];
    }
  }
};

extern "C" {

swap_status swap_sched_create(uint32_t n_gpus, const uint64_t* capacity, swap_sched_t** out) {
  if (!out || !capacity || n_gpus == 0) return SWAP_EINVAL;
  auto* s = new (std::nothrow) swap_sched();
  if (!s) return SWAP_ENOMEM;
  s->capacity.assign(capacity, capacity + n_gpus);
  *out = s;
  return SWAP_OK;
}

swap_status swap_sched_add_backend(swap_sched_t* s, uint32_t id, const uint64_t* need, int resident) {
  if (!s || !need || s->backends.count(id)) return SWAP_EINVAL;
  Backend b;
  b.need.assign(need, need + s->capacity.size());
  bool any = false;
  for (size_t g = 0; g < b.need.size(); ++g) {
    if (b.need[g] > s->capacity[g]) return SWAP_EINVAL;  // can never fit
    any |= b.need[g] > 0;
  }
  if (!any) return SWAP_EINVAL;
  if (resident) {
    for (size_t g = 0; g < b.need.size(); ++g)
      if (s->used(g) + b.need[g] > s->capacity[g]) return SWAP_ENOMEM;
  }
  b.resident = resident != 0;
  s->backends[id] = b;
  return SWAP_OK;
}

swap_status swap_sched_touch(swap_sched_t* s, uint32_t id, uint32_t queue_len, double last_access) {
  if (!s || !s->backends.count(id)) return SWAP_EINVAL;
  Backend& b = s->backends[id];
  b.queue = queue_len;
  b.last_access = last_access;
  return SWAP_OK;
}

swap_status swap_sched_lock(swap_sched_t* s, uint32_t id, int locked) {
  if (!s || !s->backends.count(id)) return SWAP_EINVAL;
  s->backends[id].locked = locked != 0;
  return SWAP_OK;
}

swap_status swap_sched_plan(const swap_sched_t* s, uint32_t id, uint32_t* victims, uint32_t cap, uint32_t* n) {
  if (!s || !n || !s->backends.count(id) || (cap && !victims)) return SWAP_EINVAL;
  std::vector<uint32_t> v;
  if (!s->plan(id, &v)) return SWAP_ENOMEM;
  *n = (uint32_t)v.size();
  if (v.size() > cap) return SWAP_EINVAL;
  std::copy(v.begin(), v.end(), victims);
  return SWAP_OK;
}

swap_status swap_sched_reserve(swap_sched_t* s, uint32_t id, double priority) {
  if (!s || !s->backends.count(id)) return SWAP_EINVAL;
  for (const auto& p : s->pending)
    if (std::get<2>(p) == id) return SWAP_ESTATE;  // already queued
  if (s->backends[id].resident) return SWAP_ESTATE;
  s->pending.insert(std::make_tuple(priority, s->seq++, id));
  return SWAP_OK;
}

swap_status swap_sched_cancel(swap_sched_t* s, uint32_t id) {
  if (!s) return SWAP_EINVAL;
  for (auto it = s->pending.begin(); it != s->pending.end(); ++it)
    if (std::get<2>(*it) == id) {
      s->pending.erase(it);
      return SWAP_OK;
    }
  return SWAP_ESTATE;
}

swap_status swap_sched_grant(swap_sched_t* s, uint32_t* id, uint32_t* victims, uint32_t cap, uint32_t* n) {
  if (!s || !id || !n || (cap && !victims)) return SWAP_EINVAL;
  *n = 0;
  if (s->pending.empty()) {
    *id = UINT32_MAX;
    return SWAP_OK;
  }
  const uint32_t head = std::get<2>(*s->pending.begin());
  *id = head;
  std::vector<uint32_t> v;
  if (!s->plan(head, &v)) return SWAP_ENOMEM;  // stays queued
  if (v.size() > cap) return SWAP_EINVAL;
  s->pending.erase(s->pending.begin());
  for (uint32_t x : v) s->backends[x].resident = false;  // release propagated on eviction
  s->backends[head].resident = true;                      // scoped acquire on every GPU of its topology
  std::copy(v.begin(), v.end(), victims);
  *n = (uint32_t)v.size();
  return SWAP_OK;
}

swap_status swap_sched_release(swap_sched_t* s, uint32_t id) {
  if (!s || !s->backends.count(id)) return SWAP_EINVAL;
  if (!s->backends[id].resident) return SWAP_ESTATE;
  s->backends[id].resident = false;
  return SWAP_OK;
}

swap_status swap_sched_query(const swap_sched_t* s, uint32_t id, int* resident, int* queued) {
  if (!s || !s->backends.count(id)) return SWAP_EINVAL;
  if (resident) *resident = s->backends.at(id).resident ? 1 : 0;
  if (queued) {
    *queued = 0;
    for (const auto& p : s->pending)
      if (std::get<2>(p) == id) *queued = 1;
  }
  return SWAP_OK;
}

swap_status swap_sched_free(const swap_sched_t* s, uint32_t gpu, uint64_t* free_bytes) {
  if (!s || !free_bytes || gpu >= s->capacity.size()) return SWAP_EINVAL;
  *free_bytes = s->capacity[gpu] - s->used(gpu);
  return SWAP_OK;
}

void swap_sched_destroy(swap_sched_t* s) { delete s; }

}  // extern "C"
