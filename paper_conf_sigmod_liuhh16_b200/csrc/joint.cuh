// joint.cuh -- the byte-JSA joint traversal of §4, kept as the
// "Joint" rung of the ablation ladder (Fig. 15):
// ibfs_run_opts.engine = IBFS_ENGINE_JOINT.  The bitwise engine (kernels.cuh) is the
// product path; this one exists to measure what the bitwise status words buy.
//
// Joint Status Array: one byte per (vertex, instance), the instances of a vertex side by
// side ("four bytes are used for each vertex"): the depth, or U = 0xff while
// unvisited.  Because a byte holds the depth itself, a level's writes (value l) are told
// apart from the previous levels' (< l) without a second copy: top-down writes l into U
// bytes; bottom-up treats a neighbour as a parent only if its byte is < l.
//
// Per level l (discovers depth l):
//   jfq_kernel   one warp per vertex scans its W status bytes and enqueues it once if any
//                active instance has it as a frontier -- top-down: byte == l - 1; bottom-up:
//                byte == U -- with __any (Fig. 4);
//   joint_expand one warp per (JFQ entry, 32-instance slice): the lanes are the instances
//                ("multiple threads with contiguous thread IDs ... the same as the number
//                of concurrently executed BFS instances"); every lane reads the
//                same adjacency entry (one broadcast load feeds all instances: the role of
//                the shared-memory cache of Fig. 5) and the neighbour's 32 status
//                bytes in one coalesced transaction.  Top-down: U -> l for the lanes whose
//                byte of the frontier is l - 1 (Fig. 5(a)); bottom-up: the frontier's byte
//                becomes l at the first neighbour with a byte < l, and the warp stops once
//                every lane is done (Fig. 5(b)).
// The host reads the per-level counters and applies the same direction policy as the
// bitwise engine (reading #7).  At the end the JSA (vertex-major) is transposed into the
// caller's instance-major int8 rows; m_s sums the degrees of the reached (vertex,
// instance) pairs.
#pragma once
#include <cstdint>

namespace ibfs {
namespace joint {

constexpr uint8_t U = 0xff;

struct JointArgs {
  const unsigned long long *off, *roff;  // out-edge rows (top-down), in-edge rows (bottom-up)
  const uint32_t *adj, *radj;
  const uint32_t *deg;
  uint32_t nva;
  int W;                  // instances per group (status bytes per vertex)
  uint8_t *jsa;           // [nva][W]
  uint32_t *jfq;          // [nva]
  unsigned long long *ctr;  // [0] |JFQ|, [1] sum of degrees of the TD frontier, [2] inspections
  uint32_t *newcnt;       // [W] discoveries per instance at this level
  uint32_t act[4];        // active instances (bit j)
};

__device__ __forceinline__ bool lane_active(const JointArgs &a, int j) { return (a.act[j >> 5] >> (j & 31)) & 1u; }

__global__ void jfq_kernel(JointArgs a, int level, int bu) {
  const int lane = threadIdx.x & 31;
  const uint32_t warps = (gridDim.x * blockDim.x) >> 5;
  const uint8_t want = bu ? U : (uint8_t)(level - 1);
  unsigned long long mf = 0;
  for (uint32_t v = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; v < a.nva; v += warps) {
    const uint8_t *row = a.jsa + (size_t)v * a.W;
    bool fr = false;
    for (int j = lane; j < a.W; j += 32) fr |= lane_active(a, j) && row[j] == want;
    if (__any_sync(0xffffffffu, fr) && lane == 0) {  // one thread enqueues
      const unsigned long long pos = atomicAdd(a.ctr, 1ull);
      a.jfq[pos] = v;
      if (!bu) mf += __ldg(a.deg + v);
    }
  }
  if (lane == 0 && mf) atomicAdd(a.ctr + 1, mf);
}

__global__ void joint_expand(JointArgs a, int level, int bu, uint32_t njfq) {
  const int lane = threadIdx.x & 31;
  const uint32_t slices = (uint32_t)a.W / 32;
  const unsigned long long items = (unsigned long long)njfq * slices;
  const unsigned long long warps = (gridDim.x * (unsigned long long)blockDim.x) >> 5;
  uint32_t found = 0, insp = 0;
  for (unsigned long long it = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5; it < items;
       it += warps) {
    const uint32_t f = a.jfq[it / slices];
    const int j = (int)(it % slices) * 32 + lane;
    uint8_t *mine = a.jsa + (size_t)f * a.W + j;
    const bool act = lane_active(a, j);
    if (!bu) {
      const bool fr = act && *mine == (uint8_t)(level - 1);
      if (!__any_sync(0xffffffffu, fr)) continue;
      const unsigned long long e0 = a.off[f], e1 = a.off[f + 1];
      for (unsigned long long e = e0; e < e1; ++e) {
        const uint32_t w = __ldg(a.adj + e);  // same address in every lane: one broadcast load
        uint8_t *st = a.jsa + (size_t)w * a.W + j;
        insp += lane == 0;
        if (fr && *st == U) {
          *st = (uint8_t)level;
          found++;
        }
      }
    } else {
      bool done = !(act && *mine == U);
      if (__all_sync(0xffffffffu, done)) continue;
      const unsigned long long e0 = a.roff[f], e1 = a.roff[f + 1];
      for (unsigned long long e = e0; e < e1; ++e) {
        if (__all_sync(0xffffffffu, done)) break;  // early termination
        const uint32_t w = __ldg(a.radj + e);
        insp += lane == 0;
        if (!done && a.jsa[(size_t)w * a.W + j] < (uint8_t)level) {  // visited before this level
          *mine = (uint8_t)level;
          done = true;
          found++;
        }
      }
    }
    if (found) { atomicAdd(a.newcnt + j, found); found = 0; }
  }
  if (insp) atomicAdd(a.ctr + 2, (unsigned long long)insp);
}

// rows[j][v] (caller ids) from the JSA: U is -1 already; isolated columns are -1.  One
// warp per (32-column tile, 32-instance slice): lane c reads column c's 32 bytes as
// 8 words, a shared-memory 32 x 32 byte transpose, lane r writes 32 bytes of row r.
__global__ void jsa_to_rows(JointArgs a, const uint32_t *tbase, const uint32_t *nzbits, uint32_t nv, int rows,
                            int8_t *out) {
  __shared__ uint32_t tile[8][32][9];  // per warp: 32 columns x 8 words (+1 pad)
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const uint32_t slices = (uint32_t)a.W / 32;
  const unsigned long long ntiles = ((unsigned long long)nv + 31) / 32;
  const unsigned long long items = ntiles * slices;
  const unsigned long long warps = (gridDim.x * (unsigned long long)blockDim.x) >> 5;
  for (unsigned long long it = (blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x) >> 5; it < items;
       it += warps) {
    const unsigned long long t = it / slices;
    const int s = (int)(it % slices);
    const unsigned long long v = t * 32 + lane;
    uint32_t wv[8];
    bool nz = false;
    uint32_t cid = 0;
    if (v < nv) {
      const uint32_t nzw = __ldg(nzbits + (v >> 5));
      nz = (nzw >> lane) & 1u;
      cid = __ldg(tbase + (v >> 7));
      for (unsigned long long k = (v >> 5) & ~3ull; k < (v >> 5); ++k) cid += __popc(__ldg(nzbits + k));
      cid += __popc(nzw & ((1u << lane) - 1u));
    }
    for (int q = 0; q < 8; ++q)
      wv[q] = nz ? *reinterpret_cast<const uint32_t *>(a.jsa + (size_t)cid * a.W + s * 32 + 4 * q) : 0xffffffffu;
    for (int q = 0; q < 8; ++q) tile[wib][lane][q] = wv[q];
    __syncwarp();
    const int r = s * 32 + lane;  // instance row this lane writes
    const unsigned long long c0 = t * 32;
    if (r < rows) {
      int8_t *dst = out + (size_t)r * nv + c0;
      const unsigned char *tb = reinterpret_cast<const unsigned char *>(&tile[wib][0][0]);
      for (int c = 0; c < 32 && c0 + c < nv; ++c)
        dst[c] = (int8_t)tb[(c * 9) * 4 + lane];  // byte `lane` of column c's 8 words
    }
    __syncwarp();
  }
}

// m_s[j] = sum over reached v of deg(v) (reading #11): thread j of a W-thread row walker.
__global__ void jsa_ms(JointArgs a, unsigned long long *m_out) {
  const int j = threadIdx.x;  // blockDim.x == W
  unsigned long long m = 0;
  for (uint32_t v = blockIdx.x; v < a.nva; v += gridDim.x)
    if (a.jsa[(size_t)v * a.W + j] != U) m += __ldg(a.deg + v);
  if (m) atomicAdd(m_out + j, m);
}

__global__ void jsa_sources(JointArgs a, const uint32_t *csrc, int rows) {
  const int j = threadIdx.x;
  if (j < rows && csrc[j] != 0xffffffffu) a.jsa[(size_t)csrc[j] * a.W + j] = 0;
}

}  // namespace joint
}  // namespace ibfs
