// plan.h -- host side of the outdegree-based GroupBy planner (§5.2).
#pragma once
#include <cstdint>
#include <functional>
#include <vector>

#include "../../include/ibfs.h"

namespace ibfs {
namespace plan {

constexpr uint32_t NO_HUB = 0xffffffffu;

// hub[r]: hub vertex of source r (NO_HUB if none), sdeg[r]: outdegree of source r,
// deg_of(x): outdegree of vertex x.  Writes the permutation to out_perm[n].
void make_plan(const ibfs_plan_params &pp, uint32_t group_bits, uint32_t n,
               const std::vector<uint32_t> &hub, const std::vector<uint32_t> &sdeg,
               const std::function<uint64_t(uint32_t)> &deg_of, uint32_t *out_perm,
               const std::vector<uint32_t> *anchor = nullptr,   // hops = 2: 2-hop anchor per source
               const std::vector<uint32_t> *hubx = nullptr);    // hops = 2: hub, or hub(m(r)) if none

// Seeded Fisher-Yates over `items` (descending i, j = mulhi64(mix64(k ^ i), i + 1),
// k = mix64(seed ^ 0x5851F42D4C957F2D)).
void seeded_shuffle(std::vector<uint32_t> &items, uint64_t seed);

}  // namespace plan
}  // namespace ibfs
