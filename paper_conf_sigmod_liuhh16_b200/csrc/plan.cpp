// plan.cpp -- outdegree-based GroupBy, §5.2.
//
//   Rule 1: both sources have outdegree < p.
//   Rule 2: both connect to a common vertex of outdegree > q.
//   q = 128, p ascending over {4, 16, 64, 128}.
//   groups satisfying both rules run directly once they reach the group size N;
//   otherwise small groups (likely from different p) are combined; finally the rest is
//   grouped "in a random manner".  P:L661: on uniform graphs share any common vertex.
// Step order (reading #16): bucket sources by hub for each p in ascending
// order, emit full W-groups per bucket (buckets visited by hub degree desc, id asc),
// then concatenate the bucket leftovers in the same order, then degree-0 sources, then a
// seeded shuffle of the remaining sources.  hub(r) is computed on the device
// (hub_kernel in ibfs.cu).  hops = 2 orders the leftovers by their 2-hop anchor (below).
#include "plan.h"

#include <algorithm>
#include <unordered_map>

namespace ibfs {
namespace plan {

static inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

void seeded_shuffle(std::vector<uint32_t> &items, uint64_t seed) {
  const uint64_t k = mix64(seed ^ 0x5851F42D4C957F2DULL);
  for (size_t i = items.size(); i-- > 1;) {
    const uint64_t j = (uint64_t)(((__uint128_t)mix64(k ^ (uint64_t)i) * (__uint128_t)(i + 1)) >> 64);
    std::swap(items[i], items[j]);
  }
}

void make_plan(const ibfs_plan_params &pp, uint32_t group_bits, uint32_t n,
               const std::vector<uint32_t> &hub, const std::vector<uint32_t> &sdeg,
               const std::function<uint64_t(uint32_t)> &deg_of, uint32_t *out_perm,
               const std::vector<uint32_t> *anchor, const std::vector<uint32_t> *hubx) {
  std::vector<uint32_t> perm;
  perm.reserve(n);
  if (pp.mode == 2) {
    for (uint32_t r = 0; r < n; ++r) perm.push_back(r);
  } else if (pp.mode == 1) {
    for (uint32_t r = 0; r < n; ++r) perm.push_back(r);
    seeded_shuffle(perm, pp.seed);
  } else {
    std::vector<uint32_t> ps(pp.p, pp.p + pp.n_p);
    std::sort(ps.begin(), ps.end());
    std::vector<char> bucketed(n, 0);
    struct Bucket { std::vector<uint32_t> items; size_t head = 0; };
    std::unordered_map<uint32_t, Bucket> buckets;
    std::vector<uint32_t> order;  // hub ids, kept sorted by (deg desc, id asc)
    auto by_degree = [&](uint32_t x, uint32_t y) {
      const uint64_t dx = deg_of(x), dy = deg_of(y);
      return dx != dy ? dx > dy : x < y;
    };
    for (uint32_t p : ps) {
      for (uint32_t r = 0; r < n; ++r) {
        if (bucketed[r] || sdeg[r] >= p || hub[r] == NO_HUB) continue;
        auto it = buckets.find(hub[r]);
        if (it == buckets.end()) {
          it = buckets.emplace(hub[r], Bucket{}).first;
          order.push_back(hub[r]);
        }
        it->second.items.push_back(r);
        bucketed[r] = 1;
      }
      std::sort(order.begin(), order.end(), by_degree);
      for (uint32_t h : order) {
        Bucket &b = buckets[h];
        while (b.items.size() - b.head >= group_bits) {
          perm.insert(perm.end(), b.items.begin() + b.head, b.items.begin() + b.head + group_bits);
          b.head += group_bits;
        }
      }
    }
    if (!anchor) {
      for (uint32_t h : order) {
        Bucket &b = buckets[h];
        perm.insert(perm.end(), b.items.begin() + b.head, b.items.end());
      }
    }
    std::vector<uint32_t> other, late;
    for (uint32_t r = 0; r < n; ++r) {
      if (bucketed[r]) continue;
      if (sdeg[r] == 0) perm.push_back(r);
      else if (anchor && (*hubx)[r] != NO_HUB) late.push_back(r);
      else other.push_back(r);
    }
    if (anchor) {
      // hops = 2 ("as long as within the first several levels"): the bucket
      // leftovers, and the remaining sources that have a hub (or reach one through their
      // max-degree neighbour m(r): hubx = hub(m(r))), ordered by their 2-hop anchor (the
      // larger of hubx(r) and hub(hubx(r)): the core vertex they reach within two or three
      // levels), then by hubx, then by position
      std::vector<uint32_t> rest;
      for (uint32_t h : order) {
        Bucket &b = buckets[h];
        rest.insert(rest.end(), b.items.begin() + b.head, b.items.end());
      }
      rest.insert(rest.end(), late.begin(), late.end());
      std::vector<uint32_t> pos(n, 0);
      for (uint32_t i = 0; i < rest.size(); ++i) pos[rest[i]] = i;
      std::stable_sort(rest.begin(), rest.end(), [&](uint32_t x, uint32_t y) {
        // sources with a 1-hop hub first; those reached through m(r) (a level later) after
        const bool lx = hub[x] == NO_HUB, ly = hub[y] == NO_HUB;
        if (lx != ly) return !lx;
        const uint32_t ax = (*anchor)[x], ay = (*anchor)[y];
        if (ax != ay) return by_degree(ax, ay);
        const uint32_t hx = (*hubx)[x], hy = (*hubx)[y];
        if (hx != hy) return by_degree(hx, hy);
        return pos[x] < pos[y];
      });
      perm.insert(perm.end(), rest.begin(), rest.end());
    }
    seeded_shuffle(other, pp.seed);
    perm.insert(perm.end(), other.begin(), other.end());
  }
  std::copy(perm.begin(), perm.end(), out_perm);
}

}  // namespace plan
}  // namespace ibfs
