// kernels.cuh -- the per-level kernels of the joint bitwise traversal (sm_100a).
//
// One group = up to W BFS instances sharing one W-bit status word per vertex (the
// Bitwise Status Array, §6).  Per group the device holds
//   visited[v]  bit j = 1 iff instance j reached v at an earlier level  (BSA_k)
//   S_l[v]      ring of R level snapshots (slot l % R): the bits discovered at level l,
//               i.e. BSA_l+1 XOR BSA_l.  S_l-1 is the top-down frontier word F of level
//               l (Alg. 2 "BSA_k+1 XOR BSA_k"); S_l accumulates level l's new bits
//               (Alg. 1).  S_0 holds the sources.
//   tdq / buq   the joint frontier queues (JFQ) of the next level, one per
//               direction, written by the commit that precedes it: top-down = vertices
//               with new bits (Alg. 2 l.3 "BSA_k+1 XOR BSA_k"), bottom-up = vertices with
//               an unvisited active bit (Alg. 2 l.7, reading #6).  Each array holds
//               "light" vertices (degree <= LIGHT_DEG) from the front and "heavy" ones
//               from the back; a shared frontier is enqueued once.
// Level l (discovers depth l; reading #20) is two launches:
//   expand_kernel<T>(l): expands the level's JFQ --
//       top-down  N[w] |= F[f] & ~visited[w]   with RED.OR (Alg. 1 l.5),
//       bottom-up acc  |= visited[w] & T[f], T = ~visited[f] & active, early exit when
//                 acc == T (Alg. 1 l.7-10; reading #5), N[f] = acc.
//   commit_kernel<T>(l): visited |= S_l ("the differences between BSA_k and
//       BSA_k+1 are used to identify the just visited vertices"), zeroes slot l+1, builds
//       both queues of level l+1 with warp ballots (the paper's __any/__ballot JFQ
//       generation), counts the direction-switch inputs; its last CTA per group
//       decides the next level's direction (reading #7).
//   depth_kernel<T>: depth[j][v] = the level l whose snapshot first holds bit j of v
//       (-1 if none), written row-major through a shared-memory transpose, once per
//       ring round (normally once per group, after the last level); also sums m_s.
// Vertices of degree > HUB_T never enter the queues: their rows are split into static
// chunks of CHUNK edges that whole CTAs sweep (the paper's shared "cache" of a
// frontier's adjacency used by all instances, as CTA-cooperative expansion).
#pragma once
#include <cstdint>
#include <cuda.h>
#include "word.cuh"

namespace ibfs {

constexpr int BLOCK = 256;
constexpr int NWARP = BLOCK / 32;
constexpr int QL = 1024;         // light-queue entries per work item
#ifndef IBFS_DEPTH_SKIP
#define IBFS_DEPTH_SKIP 1  // skip the level-0 and sparse-committed snapshots (A/B knob)
#endif
#ifndef IBFS_QH
#define IBFS_QH 64
#endif
#ifndef IBFS_QBH
#define IBFS_QBH 2048
#endif
#ifndef IBFS_LIGHT_DEG
#define IBFS_LIGHT_DEG 64
#endif
#ifndef IBFS_HUB_T
#define IBFS_HUB_T 16384
#endif
constexpr int QH = IBFS_QH;             // heavy TD-queue entries per work item
constexpr int QBH = IBFS_QBH;           // heavy BU-queue entries per work item
constexpr int LIGHT_DEG = IBFS_LIGHT_DEG;  // degree <= LIGHT_DEG: light
constexpr int HUB_T = IBFS_HUB_T;       // degree > HUB_T: hub (chunked rows)
constexpr int CHUNK = IBFS_HUB_T;       // hub-row edges per work item
constexpr int MAXL = 130;        // level index 1..129 (129 only detects depth > 127)
constexpr int MAX_G = 128;       // groups per launch batch
constexpr unsigned FULL = 0xffffffffu;
#ifndef IBFS_EXPAND_MINB
#define IBFS_EXPAND_MINB 3  // min resident expand CTAs per SM (register cap)
#endif
#ifndef IBFS_BU_U
#define IBFS_BU_U 4  // neighbours a bottom-up thread inspects per step (loads in flight)
#endif
constexpr int BU_U = IBFS_BU_U;

// queue classes
constexpr int Q_TDL = 0, Q_TDH = 1, Q_BUL = 2, Q_BUH = 3;
constexpr int Q_TDC = 4, Q_BUC = 5;  // hub-chunk queues (chunk indices, not vertices)
constexpr int NQ = 6;

struct HubChunk {
  unsigned long long e0, e1;
  uint32_t v;
  uint32_t first;
};

// Per group per level counters (device).  dir: 0 = level not run, 1 = TD, 2 = BU.
struct LevelStat {
  unsigned long long jfq, fq, proc, insp, writes, newp, nf;
  unsigned long long gath;  // neighbour status words actually gathered (BU frontier hits, TD pre-checks)
  uint32_t dir;
  uint32_t flags;    // bit 0: the depth kernel skips this level's snapshot (late list +
                     // fix-up); bit 1: the level's commit was sparse
};

template <typename T>
struct GroupCtrl {
  T active;   // instances that discovered something at the last committed level
  T newacc;   // OR of the new bits of the running commit
  unsigned long long n_f, m_f, newp;
  unsigned long long vpairs;  // (instance, vertex) pairs visited so far
  uint32_t qlen[2][NQ]; // [parity of the producing level][queue class]
  uint32_t dir;         // direction of the next expand: 0 TD, 1 BU
  uint32_t td_filter;   // top-down reads visited[w] before its RED.OR (else the commit masks)
  uint32_t done;
  uint32_t arrive;
  uint32_t last_level;
  // per-instance direction split of a bottom-up level (include/ibfs.h IBFS_SPLIT_*):
  // td_bits = the active instances expanded top-down in the next level when dir == BU
  T td_bits;
  uint32_t sparse;  // the last commit was sparse (no bottom-up queue: the next level is TD)
  // the next expand marks the 32-vertex chunks it writes (for a sparse commit): only for a
  // top-down level whose frontier edge count m_f could leave few writes (m_f <= 2 nva); a
  // heavy level (level 2 of a hub-sharing group: m_f ~ 10^8) is never sparse, and a byte
  // store per RED.OR would add a third write request to every update
  uint32_t td_mark;
  // the next bottom-up expand probes the frontier bitmap before gathering (Policy::bu_probe):
  // worth it when the frontier (vertices with new bits) is a small part of the graph, so
  // most neighbours are not in it; on a dense frontier the probe only adds latency
  uint32_t bu_probe;
  // levels whose snapshot the depth kernel does not read (bit l): level 0 (the sources,
  // written by late_fix_kernel from the source list) and every sparse-committed level,
  // whose few new vertices went to the late list instead
  unsigned long long skip_lv[2];
  float bitw[WordBits<T>::value];  // sampled degree sum of the new frontier per instance (commit)
  float cumw[WordBits<T>::value];  // running sum of bitw over the levels so far (visited edges)
};

struct Policy {
  uint32_t mode;      // IBFS_DIR_*
  uint32_t bu_from;
  float alpha, beta;
  unsigned long long nv_active;  // vertices with degree > 0
  unsigned long long ne;         // CSR entries
  uint32_t sched_len;
  uint32_t split, split_mod;  // IBFS_SPLIT_*
  float split_div;
  uint32_t max_depth;  // k-hop cap (0 = unbounded)
  uint32_t bu_probe;   // frontier-bitmap probes in BU: 0 never, 1 sparse frontiers (default), 2 always
  float split_rel;     // > 0: also top-down when m_f(j) * split_rel < max over active j' of m_f(j')
  uint32_t td_scheck;  // top-down ORs read S_l[w] first: 1 unfiltered ones, 2 all (A/B knob IBFS_TD_SCHECK)
  uint8_t sched[MAXL];  // 0 TD / 1 BU for level l at index l-1
};

template <typename T>
struct BatchArgs {
  const unsigned long long *off;  // compacted CSR (vertices of degree > 0 only): out-edges
  const uint32_t *adj;            // (top-down reads these rows)
  const uint32_t *deg;
  // in-edge CSR for bottom-up ("directed graphs also store reverse edges"); for
  // an undirected graph these alias off / adj / deg and the hub lists below
  const unsigned long long *roff;
  const uint32_t *radj;
  const uint32_t *rdeg;
  uint32_t directed;
  const uint32_t *tbase;   // [nv/128 + 1] non-isolated vertices before each 128-vertex tile
  const uint32_t *nzbits;  // [nv/32] bit v%32 of word v/32: vertex v has degree > 0
  uint32_t nv;     // vertices of the caller's graph (depth row length)
  uint32_t nva;    // non-isolated vertices (status word arrays, queues)
  size_t gstride;  // words per per-group array
  T *visited;
  T *ring;       // [R][gcap][gstride] level snapshots
  int R;         // ring slots
  int gcap;      // groups allocated per slot
  uint32_t *tdq, *buq;  // [gcap][nva] queues
  uint8_t *dirty;       // [gcap][nchunk32] 32-vertex chunk of S_l written by a top-down RED.OR
  // [gcap][nchunk32] frontier bitmap of the running level: bit v%32 of word v/32 = (S_l-1[v]
  // != 0), written by the commit of level l-1 (the init for level 1).  Bottom-up needs a
  // neighbour's word only when the neighbour is in the frontier (Lemma: visited[w] & T[f]
  // = S_l-1[w] & T[f]), so the bitmap -- nva/8 bytes per group, L2-resident --
  // filters the random status gathers.
  uint32_t *fbits;
  unsigned long long *late;  // [gcap][late_cap] (level << 32 | v) new vertices of sparse commits
  uint32_t *late_n;          // [gcap] appended entries (may exceed late_cap: then no more skips)
  uint32_t late_cap;
  uint32_t clean_ring;  // 1: every ring slot is zero at batch start and is zeroed again after
                        // its depths are written (ring_clean_kernel, late_fix_kernel), so
                        // neither init nor the commits clear slots
  uint32_t nchunk32;    // ceil(nva / 32)
  GroupCtrl<T> *ctrl;
  LevelStat *lstat;     // [G][MAXL]
  uint32_t *work_ctr;   // [MAXL]
  uint32_t *batch_done;
  uint32_t *range_err;
  int G;
  uint32_t n_total;     // sources in the whole run
  uint32_t group0;      // global index of this batch's first group
  const uint32_t *src;  // this batch's sources (caller ids), group-major, row g*W + j
  const uint32_t *csrc; // the same in compacted ids (NO_VERTEX if the source is isolated)
  int8_t *out;          // row g*W + j of this batch at out + (g*W + j) * nv
  const HubChunk *chunks;       // out-edge rows of degree > HUB_T (top-down)
  uint32_t n_chunks;
  const uint32_t *hub_vtx;     // [n_hubs] compacted ids of the vertices of degree > HUB_T, ascending
  const uint32_t *hub_chunk0;  // [n_hubs + 1] first chunk of each hub (chunks are in hub order)
  uint32_t n_hubs;
  const HubChunk *rchunks;     // the same for the in-edge rows (bottom-up)
  uint32_t n_rchunks;
  const uint32_t *rhub_vtx;
  const uint32_t *rhub_chunk0;
  uint32_t n_rhubs;
  uint32_t chq_stride;         // max(n_chunks, n_rchunks)
  uint32_t *chq;               // [gcap][2][chq_stride] hub-chunk queues (TD, BU)
  uint32_t *gbar;              // [2] grid barrier (count, generation)
  unsigned long long *tstamp;  // [MAXL][3] globaltimer: first CTA start, barrier, last CTA end
  uint32_t n_iso;       // vertices of degree 0 (nv - nva)
  Policy pol;
};

constexpr uint32_t NO_VERTEX = 0xffffffffu;

template <typename T>
__device__ __forceinline__ int group_rows(const BatchArgs<T> &a, int g) {
  constexpr int W = WordBits<T>::value;
  long long r = (long long)a.n_total - (long long)(a.group0 + g) * W;
  return r >= W ? W : (r > 0 ? (int)r : 0);
}

template <typename T>
__device__ __forceinline__ T *snap(const BatchArgs<T> &a, int g, int level) {
  return a.ring + ((size_t)(level % a.R) * a.gcap + g) * a.gstride;
}
template <typename T>
__device__ __forceinline__ T *frontier_buf(const BatchArgs<T> &a, int g, int level) {
  return snap(a, g, level - 1);
}
template <typename T>
__device__ __forceinline__ T *next_buf(const BatchArgs<T> &a, int g, int level) {
  return snap(a, g, level);
}
template <typename T>
__device__ __forceinline__ uint32_t *queue_of(const BatchArgs<T> &a, int g, int cls) {
  return (cls < Q_BUL ? a.tdq : a.buq) + (size_t)g * a.nva;
}
// entry i of queue class cls (light classes from the front, heavy from the back)
template <typename T>
__device__ __forceinline__ uint32_t queue_at(const BatchArgs<T> &a, const uint32_t *q, int cls, uint32_t i) {
  return (cls & 1) ? q[a.nva - 1 - i] : q[i];
}

// Top-down write to vertex w of group g: mark its 32-vertex chunk for the sparse commit
// (a fire-and-forget byte store; the level's write count bounds the marked chunks).
template <typename T>
__device__ __forceinline__ void mark_dirty(const BatchArgs<T> &a, int g, uint32_t w) {
  a.dirty[(size_t)g * a.nchunk32 + (w >> 5)] = 1;
}

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// 32 x 32 bit transpose across a warp (rows = lanes, columns = bit positions): on return
// bit i of lane j is bit j of lane i on entry.  Recursive block swap, 5 shuffle stages.
__device__ __forceinline__ uint32_t warp_transpose32(uint32_t x) {
  const int lane = threadIdx.x & 31;
  const uint32_t masks[5] = {0x0000ffffu, 0x00ff00ffu, 0x0f0f0f0fu, 0x33333333u, 0x55555555u};
#pragma unroll
  for (int i = 0; i < 5; ++i) {
    const int s = 16 >> i;
    const uint32_t m = masks[i];
    const uint32_t y = __shfl_xor_sync(FULL, x, s);
    x = (lane & s) ? ((x & ~m) | ((y & ~m) >> s)) : ((x & m) | ((y & m) << s));
  }
  return x;
}

// Warp-aggregated append of this lane's vertex v to queue class cls when pred holds
// (one atomic per warp per class, "__ballot()").
template <typename T>
__device__ __forceinline__ void queue_push(const BatchArgs<T> &a, int g, uint32_t *qlen, int cls,
                                           bool pred, uint32_t v) {
  const uint32_t bal = __ballot_sync(FULL, pred);
  if (!bal) return;
  const int lane = threadIdx.x & 31;
  const int leader = __ffs(bal) - 1;
  uint32_t base = 0;
  if (lane == leader) base = atomicAdd(qlen + cls, (uint32_t)__popc(bal));
  base = __shfl_sync(FULL, base, leader);
  if (pred) {
    const uint32_t i = base + __popc(bal & lanemask_lt());
    uint32_t *q = queue_of(a, g, cls);
    if (cls & 1) q[a.nva - 1 - i] = v; else q[i] = v;
  }
}

// Enqueue every chunk of hub vertex v (degree > HUB_T) into hub-chunk queue cls (Q_TDC /
// Q_BUC) when pred holds: the hub is a frontier of the next level, so its row is swept
// chunk by chunk.  Warp-cooperative (all lanes must call it): the lanes holding a hub are
// served one after the other, the whole warp writing each hub's chunk indices.
template <typename T>
__device__ __forceinline__ void push_hub_chunks(const BatchArgs<T> &a, int g, uint32_t *qlen, int cls,
                                                bool pred, uint32_t v) {
  uint32_t bal = __ballot_sync(FULL, pred);
  if (!bal) return;
  const int lane = threadIdx.x & 31;
  const bool bu = cls == Q_BUC;
  uint32_t *q = a.chq + ((size_t)g * 2 + (cls - Q_TDC)) * a.chq_stride;
  const uint32_t *hvtx = bu ? a.rhub_vtx : a.hub_vtx, *hc0 = bu ? a.rhub_chunk0 : a.hub_chunk0;
  const uint32_t nh = bu ? a.n_rhubs : a.n_hubs;
  while (bal) {
    const int src = __ffs(bal) - 1;
    bal &= bal - 1;
    const uint32_t hv = __shfl_sync(FULL, v, src);
    uint32_t c0 = 0, c1 = 0, base = 0;
    if (lane == 0) {
      uint32_t lo = 0, hi = nh;  // hub index: binary search (hubs are few and sorted)
      while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (__ldg(hvtx + mid) <= hv) lo = mid; else hi = mid;
      }
      c0 = __ldg(hc0 + lo);
      c1 = __ldg(hc0 + lo + 1);
      base = atomicAdd(qlen + cls, c1 - c0);
    }
    c0 = __shfl_sync(FULL, c0, 0);
    c1 = __shfl_sync(FULL, c1, 0);
    base = __shfl_sync(FULL, base, 0);
    for (uint32_t c = c0 + lane; c < c1; c += 32) q[base + (c - c0)] = c;
  }
}

__device__ __forceinline__ int queue_class(uint32_t d, bool bu) {
  return (bu ? Q_BUL : Q_TDL) + (d > (uint32_t)LIGHT_DEG ? 1 : 0);
}

// ------------------------------------------------------------------------- init ----
// Control words, per-level counters and the item counters (one CTA per group).  Level 1
// has closed-form Eq. 1 counters over all nv vertices (reading #23): top-down, the
// frontier is the distinct sources (sum_j |FQ_j| = rows); bottom-up, every vertex but the
// instance's own source is unvisited (sum_j |FQ_j| = rows * (nv - 1), |JFQ| = nv unless
// every source is the same vertex).  Instances whose source is isolated are finished at
// level 0: they are left out of the active mask, and a group of only such instances is
// done before level 1 (its rows are -1 except the source).
template <typename T>
__global__ void init_ctrl_kernel(BatchArgs<T> a, uint32_t first_dir) {
  constexpr int W = WordBits<T>::value;
  __shared__ uint32_t s_src[W];
  __shared__ uint32_t s_distinct;
  __shared__ T s_act;
  __shared__ unsigned long long s_msrc;
  const int g = blockIdx.x;
  const int rows = group_rows(a, g);
  LevelStat *ls = a.lstat + (size_t)g * MAXL;
  for (int l = threadIdx.x; l < MAXL; l += blockDim.x) ls[l] = LevelStat{};
  if (threadIdx.x == 0) { s_distinct = 0; s_act = wzero_value<T>(); s_msrc = 0; }
  for (int j = threadIdx.x; j < rows; j += blockDim.x) s_src[j] = a.src[(size_t)g * W + j];
  __syncthreads();
  for (int j = threadIdx.x; j < rows; j += blockDim.x) {
    bool first = true;
    for (int i = 0; i < j; ++i)
      if (s_src[i] == s_src[j]) { first = false; break; }
    if (first) atomicAdd(&s_distinct, 1u);
    const uint32_t cs = a.csrc[(size_t)g * W + j];
    if (cs != NO_VERTEX) {
      set_bit_atomic(&s_act, j);
      atomicAdd(&s_msrc, (unsigned long long)__ldg(a.deg + cs));
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    GroupCtrl<T> c;
    c.active = s_act;
    c.newacc = wzero_value<T>();
    c.n_f = c.m_f = c.newp = 0;
    c.vpairs = (unsigned long long)wpopc(s_act);
    for (int p = 0; p < 2; ++p)
      for (int k = 0; k < NQ; ++k) c.qlen[p][k] = 0;
    c.dir = first_dir;
    c.td_filter = 0;
    c.td_mark = s_msrc <= 2ull * a.nva ? 1u : 0u;  // level 1's frontier edges: the sources' rows
    c.bu_probe = a.pol.bu_probe != 0 ? 1u : 0u;    // level 1's frontier: the sources
    const bool done = rows == 0 || wzero(s_act);
    c.done = done ? 1u : 0u;
    c.arrive = 0;
    c.last_level = done ? 0xffffffffu : 0u;  // done at init: no snapshot was ever written
    c.td_bits = wzero_value<T>();
    c.sparse = 0;
    c.skip_lv[0] = IBFS_DEPTH_SKIP ? 1ull : 0ull;  // level 0: the sources (late_fix_kernel)
    c.skip_lv[1] = 0ull;
    for (int j = 0; j < W; ++j) c.bitw[j] = c.cumw[j] = 0.f;
    a.ctrl[g] = c;
    if (rows > 0) {
      LevelStat *l1 = ls + 1;
      if (first_dir == 0) {
        l1->jfq = s_distinct;
        l1->fq = (unsigned long long)rows;
      } else {
        l1->jfq = (unsigned long long)a.nv - (s_distinct == 1 ? 1u : 0u);
        l1->fq = (unsigned long long)rows * ((unsigned long long)a.nv - 1ull);
      }
      if (done) {  // level 1 "runs" and finds nothing; no snapshot is read for it
        l1->dir = first_dir + 1;
        l1->flags = 1u;
      }
    }
    if (done) atomicAdd(a.batch_done, 1u);
  }
  if (g == 0)
    for (int l = threadIdx.x; l < MAXL; l += blockDim.x) {
      a.work_ctr[l] = 0;
      a.tstamp[(size_t)l * 3] = ~0ull;  // level kernels atomicMin their start here
      a.tstamp[(size_t)l * 3 + 1] = 0;
      a.tstamp[(size_t)l * 3 + 2] = 0;
    }
}

// Zero the group's visited words and the snapshot slots of levels 0 and 1 (a2; with the
// clean ring they are zero already: ms_kernel / the clean-up passes left them so); when
// level 1 runs bottom-up, enqueue every vertex of degree <= HUB_T (all are unvisited for
// some active instance unless they are the source of every active instance -- the
// expand skips those).
template <typename T>
__global__ void __launch_bounds__(BLOCK) init_state_kernel(BatchArgs<T> a, uint32_t first_dir) {
  const int g = blockIdx.y;
  if (a.ctrl[g].done) return;
  const size_t stride = (size_t)gridDim.x * BLOCK;
  const T z = wzero_value<T>();
  T *vis = a.visited + (size_t)g * a.gstride;
  T *s0 = snap(a, g, 0);
  T *s1 = snap(a, g, 1);
  uint32_t *qlen = a.ctrl[g].qlen[0];
  const size_t nvr = ((size_t)a.nva + 31) & ~(size_t)31;  // warp-uniform trip count
  for (size_t v = (size_t)blockIdx.x * BLOCK + threadIdx.x; v < nvr; v += stride) {
    const bool in = v < a.nva;
    if (in) {
      if (!a.clean_ring) {  // clean ring: visited and the slots are zero already
        st(vis + v, z);
        st(s0 + v, z);
        st(s1 + v, z);
      }
      if ((v & 31) == 0) {
        a.dirty[(size_t)g * a.nchunk32 + (v >> 5)] = 0;
        a.fbits[(size_t)g * a.nchunk32 + (v >> 5)] = 0u;
      }
    }
    if (first_dir) {
      const uint32_t d = in ? __ldg(a.rdeg + v) : 0u;  // bottom-up reads in-edge rows
      const bool q = in && d > 0 && d <= (uint32_t)HUB_T;
      queue_push(a, g, qlen, Q_BUL, q && d <= (uint32_t)LIGHT_DEG, (uint32_t)v);
      queue_push(a, g, qlen, Q_BUH, q && d > (uint32_t)LIGHT_DEG, (uint32_t)v);
      push_hub_chunks(a, g, qlen, Q_BUC, in && d > (uint32_t)HUB_T, (uint32_t)v);
    }
  }
}

// Sources: visited[s_j] |= bit j, S_0[s_j] |= bit j (depth 0) for the non-isolated
// sources; the distinct ones of degree <= HUB_T form the top-down queue of level 1.
template <typename T>
__global__ void init_sources_kernel(BatchArgs<T> a, uint32_t first_dir) {
  constexpr int W = WordBits<T>::value;
  __shared__ uint32_t s_src[W];
  const int g = blockIdx.x;
  const int rows = group_rows(a, g);
  if (rows == 0 || a.ctrl[g].done) return;
  T *vis = a.visited + (size_t)g * a.gstride;
  T *f = snap(a, g, 0);  // frontier of level 1
  for (int j = threadIdx.x; j < rows; j += blockDim.x) s_src[j] = a.csrc[(size_t)g * W + j];
  __syncthreads();
  uint32_t *qlen = a.ctrl[g].qlen[0];
  for (int j = threadIdx.x; j < W; j += blockDim.x) {  // warp-uniform loop
    bool first = false;
    uint32_t s = 0, d = 0;
    if (j < rows && s_src[j] != NO_VERTEX) {
      s = s_src[j];
      set_bit_atomic(vis + s, j);
      set_bit_atomic(f + s, j);
      atomicOr(a.fbits + (size_t)g * a.nchunk32 + (s >> 5), 1u << (s & 31));
      first = true;
      for (int i = 0; i < j; ++i)
        if (s_src[i] == s) { first = false; break; }
      d = __ldg(a.deg + s);
    }
    const bool q = first && d <= (uint32_t)HUB_T && first_dir == 0;
    queue_push(a, g, qlen, Q_TDL, q && d <= (uint32_t)LIGHT_DEG, s);
    queue_push(a, g, qlen, Q_TDH, q && d > (uint32_t)LIGHT_DEG, s);
    push_hub_chunks(a, g, qlen, Q_TDC, first && d > (uint32_t)HUB_T && first_dir == 0, s);
  }
}

// ----------------------------------------------------------------------- expand ----
struct ExpandSmem {  // static part
  uint32_t wsum[NWARP];
  uint32_t cnt[2];
  uint32_t item;
  uint32_t flag;
  uint32_t pre[3 * MAX_G * 2 + 1];   // item prefix over (phase, group, direction)
  unsigned long long acc[MAX_G][6];  // jfq, fq, proc, insp, writes, gath
};

// Dynamic part: the CTA-local copy of one work item's queue entries.
template <typename T>
struct TileQueue {
  unsigned long long start[QL];  // adjacency row start of entry i
  T word[QL];                    // TD: frontier word F; BU: target T
  uint32_t aux[QL + 1];          // degrees, then their exclusive prefix
  uint32_t vtx[QL];
};

// Exclusive scan of s[0..n) in place (n <= QL), s[n] = total.  Block-wide.
__device__ __forceinline__ void block_exclusive_scan(uint32_t *s, uint32_t n, uint32_t *wsum) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int PER = QL / BLOCK;  // 4 consecutive entries per thread
  uint32_t x[PER];
  uint32_t sum = 0;
#pragma unroll
  for (int k = 0; k < PER; ++k) {
    uint32_t i = tid * PER + k;
    x[k] = i < n ? s[i] : 0u;
    sum += x[k];
  }
  uint32_t inc = sum;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    uint32_t y = __shfl_up_sync(FULL, inc, d);
    if (lane >= d) inc += y;
  }
  if (lane == 31) wsum[warp] = inc;
  __syncthreads();
  if (warp == 0) {
    uint32_t w = lane < NWARP ? wsum[lane] : 0u;
    uint32_t wi = w;
#pragma unroll
    for (int d = 1; d < NWARP; d <<= 1) {
      uint32_t y = __shfl_up_sync(FULL, wi, d);
      if (lane >= d) wi += y;
    }
    if (lane < NWARP) wsum[lane] = wi - w;  // exclusive warp offsets
  }
  __syncthreads();
  uint32_t run = wsum[warp] + inc - sum;
#pragma unroll
  for (int k = 0; k < PER; ++k) {
    uint32_t i = tid * PER + k;
    if (i < n) s[i] = run;
    run += x[k];
  }
  if (tid == BLOCK - 1) s[n] = run;  // last thread holds the grand total
  __syncthreads();
}

// Largest q in [0, n) with s[q] <= e (s strictly increasing on the queued entries).
__device__ __forceinline__ uint32_t lbs_search(const uint32_t *s, uint32_t n, uint32_t e) {
  uint32_t lo = 0, hi = n;
  while (hi - lo > 1) {
    uint32_t mid = (lo + hi) >> 1;
    if (s[mid] <= e) lo = mid; else hi = mid;
  }
  return lo;
}

__device__ __forceinline__ void flush_counts(ExpandSmem &sm, int g, uint32_t jfq, uint32_t fq,
                                             uint32_t proc, uint32_t insp, uint32_t writes, uint32_t gath) {
  jfq = __reduce_add_sync(FULL, jfq);
  fq = __reduce_add_sync(FULL, fq);
  proc = __reduce_add_sync(FULL, proc);
  insp = __reduce_add_sync(FULL, insp);
  writes = __reduce_add_sync(FULL, writes);
  gath = __reduce_add_sync(FULL, gath);
  if ((threadIdx.x & 31) == 0) {
    if (jfq) atomicAdd(&sm.acc[g][0], (unsigned long long)jfq);
    if (fq) atomicAdd(&sm.acc[g][1], (unsigned long long)fq);
    if (proc) atomicAdd(&sm.acc[g][2], (unsigned long long)proc);
    if (insp) atomicAdd(&sm.acc[g][3], (unsigned long long)insp);
    if (writes) atomicAdd(&sm.acc[g][4], (unsigned long long)writes);
    if (gath) atomicAdd(&sm.acc[g][5], (unsigned long long)gath);
  }
}

// Top-down item: entries [i0, i1) of a TD queue class.  The frontier words and rows of
// the entries are staged in shared memory, then an edge-balanced sweep (load-balanced
// search on the degree prefix) ORs each frontier word into its unvisited neighbours
// (Alg. 1 l.4-5): consecutive threads read consecutive adjacency entries.
// fmask: the instances expanded top-down (all of them in a TD level, td_bits in a split
// BU level); entries whose frontier word has none of them sweep no edges.
template <typename T>
__device__ void item_td(const BatchArgs<T> &a, ExpandSmem &sm, TileQueue<T> &tq, int g, int cls,
                        uint32_t i0, uint32_t i1, int level, bool filt, T fmask, bool mark) {
  const int tid = threadIdx.x;
  const T *F = frontier_buf(a, g, level);
  T *N = next_buf(a, g, level);
  const T *vis = a.visited + (size_t)g * a.gstride;
  const uint32_t *q = queue_of(a, g, cls);
  const uint32_t qn = i1 - i0;
  uint32_t insp = 0, writes = 0, gath = 0;
  for (uint32_t i = tid; i < qn; i += BLOCK) {
    const uint32_t v = queue_at(a, q, cls, i0 + i);
    const T f = wand(ldg(F + v), fmask);
    tq.start[i] = __ldg(a.off + v);
    tq.word[i] = f;
    tq.aux[i] = wzero(f) ? 0u : __ldg(a.deg + v);
  }
  __syncthreads();
  block_exclusive_scan(tq.aux, qn, sm.wsum);
  const uint32_t total = tq.aux[qn];
  constexpr int U = 4;
  for (uint32_t e0 = 0; e0 < total; e0 += BLOCK * U) {
    uint32_t w[U];
    T fw[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t e = e0 + u * BLOCK + tid;
      w[u] = 0xffffffffu;
      if (e < total) {
        const uint32_t k = lbs_search(tq.aux, qn, e);
        w[u] = __ldg(a.adj + tq.start[k] + (e - tq.aux[k]));
        fw[u] = tq.word[k];
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (w[u] != 0xffffffffu) {
        insp++;
        gath += filt ? 1u : 0u;
        T b = filt ? wandn(fw[u], ldg(vis + w[u])) : fw[u];
        // IBFS_TD_SCHECK: skip the RED.OR when S_l[w] already holds the bits (an L2 read
        // instead of a read-modify-write; a stale read shows a subset of the bits, so a
        // needed OR is never skipped)
        if (a.pol.td_scheck > (filt ? 1u : 0u) && !wzero(b)) b = wandn(b, ldcg_w(N + w[u]));
        if (!wzero(b)) {
          red_or(N + w[u], b);
          writes++;
          if (mark) mark_dirty(a, g, w[u]);
        }
      }
    }
  }
  flush_counts(sm, g, 0u, 0u, tid == 0 ? qn : 0u, insp, writes, gath);
}

// Bottom-up item: entries [i0, i1) of a BU queue class.
// Every entry f with T = active & ~visited[f] != 0 is a frontier (Alg. 2 l.7, reading
// #6); it ORs its neighbours' visited words masked by T in CSR order and stops once the
// accumulated word covers T (early termination, active mask of reading #5).  One
// thread owns one frontier at a time ("a single thread to work on each frontier",
// P:L813) and inspects 4 neighbours per step, with the next step's adjacency loads in
// flight during this step's gathers; each warp refills its lanes from a private ring as
// soon as a frontier terminates, so lanes stay busy until the item drains.
template <typename T>
struct BuRing {  // per-warp rings of QL / NWARP entries, carved from TileQueue storage
  unsigned long long start[QL];
  T word[QL];
  uint32_t deg[QL];
  uint32_t vtx[QL];
};

template <typename T>
// active: the group's active instances (Eq. 1 counters, reading #23); td_bits: those a
// split level expands top-down instead (excluded from T; N[f] is then shared with the
// top-down part, so the result is ORed in rather than stored).
__device__ void item_bu(const BatchArgs<T> &a, ExpandSmem &sm, TileQueue<T> &tq, int g, int cls,
                        uint32_t i0, uint32_t i1, int level, T active, T td_bits, bool probe) {
  constexpr int QW = QL / NWARP;  // ring entries per warp (128)
  static_assert(sizeof(BuRing<T>) <= sizeof(TileQueue<T>), "BU ring must fit the item storage");
  BuRing<T> &bq = *reinterpret_cast<BuRing<T> *>(&tq);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  T *N = next_buf(a, g, level);
  const T *vis = a.visited + (size_t)g * a.gstride;
  const T *F = frontier_buf(a, g, level);                 // S_l-1: the neighbours' new bits
  const uint32_t *fb = a.fbits + (size_t)g * a.nchunk32;  // its nonzero bitmap
  const uint32_t *q = queue_of(a, g, cls);
  uint32_t jfq = 0, fq = 0, proc = 0, insp = 0, writes = 0, gath = 0;
  const bool split = !wzero(td_bits);
  if (tid == 0) sm.cnt[0] = i0;
  __syncthreads();
  const int qbase = warp * QW;
  uint32_t head = 0, tail = 0;  // warp-uniform ring cursors
  bool range_done = false;
  bool has = false;
  uint32_t v = 0, d = 0, k = 0;
  unsigned long long s0 = 0;
  T tg = wzero_value<T>(), acc = wzero_value<T>();
  // software pipeline over a row, BU_U neighbours per step: the step's ids and their
  // frontier-bitmap words are in (wn, mn); the next step's ids in wn2 (prefetched); the
  // bitmap words of step s + 1 are loaded during step s
  uint32_t wn[BU_U], mn[BU_U], wn2[BU_U];
  // refill pipeline: the loads for the next 32 queue entries are issued one round early
  uint32_t c_next = 0, x_next = 0, dx_next = 0;
  T tx_next = wzero_value<T>();
  unsigned long long ox_next = 0;
  auto issue_refill = [&]() {
    if (lane == 0) c_next = atomicAdd(&sm.cnt[0], 32u);
    c_next = __shfl_sync(FULL, c_next, 0);
    const uint32_t i = c_next + lane;
    if (c_next < i1 && i < i1) {
      x_next = queue_at(a, q, cls, i);
      tx_next = wandn(active, ldg(vis + x_next));
      dx_next = __ldg(a.rdeg + x_next);
      ox_next = __ldg(a.roff + x_next);
    } else {
      tx_next = wzero_value<T>();
      dx_next = 0;
    }
  };
  issue_refill();
  for (;;) {
    if (!range_done && tail - head <= (uint32_t)(QW - 32)) {
      if (c_next >= i1) {
        range_done = true;
      } else {
        const T tfull = tx_next;
        const T tx = wandn(tfull, td_bits);
        const bool keep = !wzero(tx);
        if (!wzero(tfull) && level > 1) { jfq++; fq += wpopc(tfull); }  // level 1: closed form (init)
        const uint32_t bal = __ballot_sync(FULL, keep);
        if (keep) {
          const uint32_t pos = qbase + ((tail + __popc(bal & lanemask_lt())) & (QW - 1));
          bq.start[pos] = ox_next;
          bq.word[pos] = tx;
          bq.deg[pos] = dx_next;
          bq.vtx[pos] = x_next;
        }
        tail += __popc(bal);
        __syncwarp();
        issue_refill();
      }
    }
    const uint32_t idle = __ballot_sync(FULL, !has);
    const uint32_t avail = tail - head;
    if (!has) {
      const uint32_t r = __popc(idle & lanemask_lt());
      if (r < avail) {
        const uint32_t pos = qbase + ((head + r) & (QW - 1));
        s0 = bq.start[pos];
        tg = bq.word[pos];
        d = bq.deg[pos];
        v = bq.vtx[pos];
        k = 0;
        acc = wzero_value<T>();
        has = true;
        proc++;
#pragma unroll
        for (int u = 0; u < BU_U; ++u) wn[u] = ((uint32_t)u < d) ? __ldg(a.radj + s0 + u) : 0xffffffffu;
#pragma unroll
        for (int u = 0; u < BU_U; ++u) wn2[u] = ((uint32_t)(BU_U + u) < d) ? __ldg(a.radj + s0 + BU_U + u) : 0xffffffffu;
        // the first step gathers without the bitmap probe: most vertices stop within their
        // first neighbours (hub-first rows, frontier hubs), and a probe there would put an
        // L2 round trip on every vertex's critical path
#pragma unroll
        for (int u = 0; u < BU_U; ++u) mn[u] = 0xffffffffu;
      }
    }
    head += min((uint32_t)__popc(idle), avail);
    __syncwarp();
    const uint32_t busy = __ballot_sync(FULL, has);
    if (!busy) {
      if (range_done && head == tail) break;
      continue;
    }
    if (has) {
      // neighbour w contributes visited[w] & T = S_l-1[w] & T (a bit of T visited at w
      // before level l-1 would have reached f already): gather S_l-1[w] only when w is in
      // the frontier bitmap
      T x[BU_U];
#pragma unroll
      for (int u = 0; u < BU_U; ++u) {
        const bool hit = wn[u] != 0xffffffffu && ((mn[u] >> (wn[u] & 31)) & 1u);
        x[u] = hit ? ldg(F + wn[u]) : wzero_value<T>();
        gath += hit ? 1u : 0u;
        insp += wn[u] != 0xffffffffu ? 1u : 0u;
      }
      k += BU_U;
#pragma unroll
      for (int u = 0; u < BU_U; ++u) wn[u] = wn2[u];
#pragma unroll
      for (int u = 0; u < BU_U; ++u) mn[u] = (probe && wn[u] != 0xffffffffu) ? __ldg(fb + (wn[u] >> 5)) : 0xffffffffu;
#pragma unroll
      for (int u = 0; u < BU_U; ++u) wn2[u] = (k + BU_U + u < d) ? __ldg(a.radj + s0 + k + BU_U + u) : 0xffffffffu;
#pragma unroll
      for (int u = 0; u < BU_U; ++u) acc = wor(acc, wand(x[u], tg));
      if (weq(acc, tg) || k >= d) {
        if (!wzero(acc)) {
          if (split) red_or(N + v, acc); else st(N + v, acc);
          writes++;
        }
        has = false;
      }
    }
  }
  flush_counts(sm, g, jfq, fq, proc, insp, writes, gath);
}

// Hub chunk, top-down: CHUNK edges of one hub's row swept by the whole CTA.
template <typename T>
__device__ void hub_td(const BatchArgs<T> &a, ExpandSmem &sm, int g, const HubChunk c, int level, bool filt,
                       T fmask, bool mark) {
  const int tid = threadIdx.x;
  const T *F = frontier_buf(a, g, level);
  T *N = next_buf(a, g, level);
  const T *vis = a.visited + (size_t)g * a.gstride;
  const T f = wand(ldg(F + c.v), fmask);
  if (wzero(f)) return;
  uint32_t insp = 0, writes = 0, gath = 0;
  constexpr int U = 8;
  for (unsigned long long e0 = c.e0; e0 < c.e1; e0 += BLOCK * U) {
    uint32_t w[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const unsigned long long e = e0 + u * BLOCK + tid;
      w[u] = e < c.e1 ? __ldg(a.adj + e) : 0xffffffffu;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (w[u] != 0xffffffffu) {
        insp++;
        gath += filt ? 1u : 0u;
        T b = filt ? wandn(f, ldg(vis + w[u])) : f;
        if (a.pol.td_scheck > (filt ? 1u : 0u) && !wzero(b)) b = wandn(b, ldcg_w(N + w[u]));
        if (!wzero(b)) {
          red_or(N + w[u], b);
          writes++;
          if (mark) mark_dirty(a, g, w[u]);
        }
      }
    }
  }
  const bool first = c.first && tid == 0;
  flush_counts(sm, g, 0u, 0u, first ? 1u : 0u, insp, writes, gath);
}

// Hub chunk, bottom-up: the CTA ORs a chunk of the hub's neighbours in waves, with a
// block OR-reduce and an exit test per wave against T and the bits other chunks have
// already found (atomically accumulated in N[hub]).
template <typename T>
__device__ void hub_bu(const BatchArgs<T> &a, ExpandSmem &sm, T *s_red, int g, const HubChunk c,
                       int level, T active, T td_bits, bool probe) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  T *N = next_buf(a, g, level);
  const T *vis = a.visited + (size_t)g * a.gstride;
  const T *F = frontier_buf(a, g, level);
  const uint32_t *fb = a.fbits + (size_t)g * a.nchunk32;
  const T tfull = wandn(active, ldg(vis + c.v));
  const T tg = wandn(tfull, td_bits);
  const bool first = c.first && tid == 0;
  const bool cnt = first && level > 1 && !wzero(tfull);  // level 1: closed form (init)
  if (wzero(tg)) {
    flush_counts(sm, g, cnt ? 1u : 0u, cnt ? (uint32_t)wpopc(tfull) : 0u, 0u, 0u, 0u, 0u);
    return;
  }
  if (tid == 0) sm.flag = weq(wand(ldv(N + c.v), tg), tg) ? 1u : 0u;
  __syncthreads();
  uint32_t insp = 0, writes = 0, gath = 0;
  T acc = wzero_value<T>();
  if (!sm.flag) {
    constexpr int U = 4;
    for (unsigned long long e0 = c.e0; e0 < c.e1; e0 += BLOCK * U) {
      T x = wzero_value<T>();
      uint32_t w[U], m[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const unsigned long long e = e0 + u * BLOCK + tid;
        w[u] = e < c.e1 ? __ldg(a.radj + e) : 0xffffffffu;
      }
      // the first wave (the row's highest-degree neighbours) gathers directly; later waves
      // probe the frontier bitmap first
#pragma unroll
      for (int u = 0; u < U; ++u)
        m[u] = (e0 == c.e0 || !probe) ? 0xffffffffu : (w[u] != 0xffffffffu ? __ldg(fb + (w[u] >> 5)) : 0u);
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (w[u] != 0xffffffffu) {
          insp++;
          if ((m[u] >> (w[u] & 31)) & 1u) {  // frontier neighbour: S_l-1[w] & T (see item_bu)
            x = wor(x, wand(ldg(F + w[u]), tg));
            gath++;
          }
        }
      }
      x = warp_or(x);
      if (lane == 0) s_red[warp] = x;
      __syncthreads();
#pragma unroll
      for (int k = 0; k < NWARP; ++k) acc = wor(acc, s_red[k]);
      if (tid == 0) sm.flag = weq(wand(wor(acc, ldv(N + c.v)), tg), tg) ? 1u : 0u;
      __syncthreads();
      if (sm.flag) break;
    }
    if (tid == 0 && !wzero(acc)) { red_or(N + c.v, acc); writes++; }
  }
  flush_counts(sm, g, cnt ? 1u : 0u, cnt ? (uint32_t)wpopc(tfull) : 0u, first ? 1u : 0u, insp, writes, gath);
}

// Expand phase of level `level` for all groups of a batch.  Work items, pulled by CTAs
// from a per-level counter, in three phases -- frontier hub chunks, then heavy-queue
// items, then light-queue items -- each carrying its group and direction.  A group runs
// its top-down part when its level is TD or a split BU level (td_bits != 0), and its
// bottom-up part when the level is BU.  The control words were written by the commit
// phase of this launch (before the grid barrier): read them through L2 (ld.cg).
template <typename T>
__device__ void expand_phase(const BatchArgs<T> &a, int level, ExpandSmem &sm, T *s_red, TileQueue<T> &tq) {
  const int tid = threadIdx.x;
  for (int i = tid; i < a.G * 6; i += BLOCK) sm.acc[i / 6][i % 6] = 0ull;
  const int par = (level - 1) & 1;  // queues were produced by commit l-1 (or init)
  const int nslot = 3 * a.G * 2;
  for (int i = tid; i < nslot; i += BLOCK) {  // items of slot (phase, group, direction)
    const int ph = i / (2 * a.G), g = (i >> 1) % a.G, d = i & 1;
    const GroupCtrl<T> *c = a.ctrl + g;
    uint32_t n = 0;
    if (!ldcg(&c->done)) {
      const uint32_t dir = ldcg(&c->dir);
      const bool on = d ? dir == 1 : (dir == 0 || !wzero(ldcg_w(&c->td_bits)));
      if (on) {
        const int base = d ? Q_BUL : Q_TDL;
        const uint32_t *ql = c->qlen[par];
        if (ph == 0) n = ldcg(ql + (d ? Q_BUC : Q_TDC));
        else if (ph == 1) { const uint32_t per = d ? QBH : QH; n = (ldcg(ql + base + 1) + per - 1) / per; }
        else n = (ldcg(ql + base) + QL - 1) / QL;
      }
    }
    sm.pre[i] = n;
  }
  __syncthreads();
  if (tid < 32) {  // exclusive prefix over the <= 6 * MAX_G slots: lane-contiguous segments
    const int seg = (nslot + 31) / 32, i0 = min(tid * seg, nslot), i1 = min(i0 + seg, nslot);
    uint32_t sum = 0;
    for (int i = i0; i < i1; ++i) sum += sm.pre[i];
    uint32_t inc = sum;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(FULL, inc, d);
      if (tid >= d) inc += y;
    }
    uint32_t run = inc - sum;
    for (int i = i0; i < i1; ++i) { const uint32_t x = sm.pre[i]; sm.pre[i] = run; run += x; }
    if (tid == 31) sm.pre[nslot] = inc;
  }
  __syncthreads();
  const uint32_t total = sm.pre[nslot];
  uint32_t pending = 0;
  if (tid == 0) pending = atomicAdd(a.work_ctr + level, 1u);
  for (;;) {
    __syncthreads();
    if (tid == 0) {
      sm.item = pending;
      if (pending < total) pending = atomicAdd(a.work_ctr + level, 1u);
    }
    __syncthreads();
    const uint32_t item = sm.item;
    if (item >= total) break;
    uint32_t lo = 0, hi = (uint32_t)nslot;  // the slot with pre[lo] <= item < pre[lo + 1]
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (sm.pre[mid] <= item) lo = mid; else hi = mid;
    }
    const int ph = (int)lo / (2 * a.G), g = (int)(lo >> 1) % a.G, d = (int)(lo & 1);
    const uint32_t k = item - sm.pre[lo];
    const GroupCtrl<T> *c = a.ctrl + g;
    const bool bu_level = ldcg(&c->dir) == 1;
    const T td_bits = bu_level ? ldcg_w(&c->td_bits) : wzero_value<T>();
    const T all = wnot(wzero_value<T>());
    // the top-down part of a split bottom-up level expands instances that are still early
    // in their traversal (most targets unvisited for them): no visited pre-check gather,
    // the RED.ORs go out directly (the commit masks bits that were already visited)
    const bool filt = !bu_level && ldcg(&c->td_filter) != 0;
    const bool mark = !bu_level && ldcg(&c->td_mark) != 0;
    const bool probe = ldcg(&c->bu_probe) != 0;
    if (ph == 0) {
      const uint32_t ci = a.chq[((size_t)g * 2 + d) * a.chq_stride + k];
      const HubChunk hc = d ? a.rchunks[ci] : a.chunks[ci];
      if (d == 0) hub_td<T>(a, sm, g, hc, level, filt, bu_level ? td_bits : all, mark);
      else hub_bu<T>(a, sm, s_red, g, hc, level, ldcg_w(&c->active), td_bits, probe);
      continue;
    }
    const bool heavy = ph == 1;
    const int cls = (d ? Q_BUL : Q_TDL) + (heavy ? 1 : 0);
    const uint32_t qlen = ldcg(c->qlen[par] + cls);
    const uint32_t per = d ? (heavy ? QBH : QL) : (heavy ? QH : QL);
    const uint32_t i0 = k * per, i1 = min(qlen, i0 + per);
    if (d == 0) item_td<T>(a, sm, tq, g, cls, i0, i1, level, filt, bu_level ? td_bits : all, mark);
    else item_bu<T>(a, sm, tq, g, cls, i0, i1, level, ldcg_w(&c->active), td_bits, probe);
  }
  __syncthreads();
  for (int i = tid; i < a.G; i += BLOCK) {
    LevelStat *ls = a.lstat + (size_t)i * MAXL + level;
    if (sm.acc[i][0]) atomicAdd(&ls->jfq, sm.acc[i][0]);
    if (sm.acc[i][1]) atomicAdd(&ls->fq, sm.acc[i][1]);
    if (sm.acc[i][2]) atomicAdd(&ls->proc, sm.acc[i][2]);
    if (sm.acc[i][3]) atomicAdd(&ls->insp, sm.acc[i][3]);
    if (sm.acc[i][4]) atomicAdd(&ls->writes, sm.acc[i][4]);
    if (sm.acc[i][5]) atomicAdd(&ls->gath, sm.acc[i][5]);
  }
}

// ----------------------------------------------------------------------- commit ----
__device__ __forceinline__ unsigned long long warp_sum64(unsigned long long x) {
  uint32_t lo = (uint32_t)x, hi = (uint32_t)(x >> 32);
  // exact 64-bit sum via 16-bit limbs (no u32 overflow for 32 lanes)
  unsigned long long s0 = __reduce_add_sync(FULL, lo & 0xffffu);
  unsigned long long s1 = __reduce_add_sync(FULL, lo >> 16);
  unsigned long long s2 = __reduce_add_sync(FULL, hi & 0xffffu);
  unsigned long long s3 = __reduce_add_sync(FULL, hi >> 16);
  return s0 + (s1 << 16) + (s2 << 32) + (s3 << 48);
}

__device__ __forceinline__ bool decide_bu(const Policy &p, uint32_t next_level, uint32_t cur_dir,
                                          unsigned long long n_f, unsigned long long m_f) {
  if (p.mode == 1) return false;
  if (p.mode == 2) return next_level >= p.bu_from;
  if (p.mode == 3 && next_level - 1 < p.sched_len) return p.sched[next_level - 1] != 0;
  // auto (reading #7): TD -> BU when the edges of the next frontier, m_f,
  // exceed ne / alpha (in joint BFS nearly every vertex keeps an unvisited active bit
  // for several levels, so Beamer's unexplored-edge count m_u is ~ne); BU -> TD when the
  // frontier holds fewer than nv_active / beta vertices.
  if (cur_dir == 0) return m_f > 0 && (double)m_f * (double)p.alpha > (double)p.ne;
  return !((double)n_f * (double)p.beta < (double)p.nv_active);
}

// Commit of level l for one group (blockIdx.y): visited |= S_l, zero slot l+1, and
// build both JFQs of level l+1 -- top-down: vertices with new bits; bottom-up: vertices
// with an unvisited bit of an instance active before this level (a superset of the
// active set after it: the expand masks with the final one, Lemma C3.5).
template <typename T>
struct CommitSmem {
  unsigned long long red[NWARP][3];
  T orr[NWARP];
  uint32_t last;
  uint32_t wcnt[NWARP][4];
  uint32_t qbase[4];
  float bcnt[WordBits<T>::value];       // sampled per-instance frontier degree sums of this CTA
  uint32_t tdb[WordBits<T>::value / 32];  // split decision (last CTA of a group)
  uint32_t wmax;                           // max sampled m_f(j) over active j (float bits)
};

// Per-instance frontier edge counts m_f(j) for the split decision (IBFS_SPLIT_AUTO) are
// sampled: the first vertex of each thread in every SAMPLE_TILES-th commit tile, i.e.
// 1 / SAMPLE of the vertices.  A warp transposes its 32 sampled new-bit words (lane i
// then holds the mask M of sampled vertices new for instance 32p + i) and weights them
// by degree through the degree bit planes D_b = ballot(bit b of deg): sum_b popc(M & D_b) << b.
constexpr int SAMPLE_TILES = 4;
constexpr int SPLIT_HEAVY = 1024;  // frontier vertices above this degree are counted exactly

// Commit of level lc for one tile of group g: the CVT * BLOCK vertices from `base`.
// visited |= S_lc, zero slot lc + 1, build both JFQs of level lc + 1 -- top-down: vertices
// with new bits; bottom-up: vertices with an unvisited bit of an instance active before
// this level (a superset of the active set after it: the expand masks with the final
// one, Lemma C3.5); hubs go to the hub-chunk queues.  The four vertex-queue classes are
// appended with one atomic per class per tile (block-wide ballot prefix).  Counters
// (n_f, m_f, new pairs, OR of new bits) accumulate in the caller's registers.
constexpr int CVT = 4;
constexpr int CTILE = CVT * BLOCK;  // vertices per commit tile
constexpr int SAMPLE = SAMPLE_TILES * CVT;

// Sparse commit of level lc: after a pure top-down level whose writes
// touched at most a quarter of the 32-vertex chunks, the commit reads S_l / visited /
// degrees only in the chunks marked dirty (every other chunk of S_l is zero: nothing new
// there) and builds no bottom-up queue, so the next level must run top-down -- allowed
// in auto mode (the override is a performance choice, never a result change) and in a
// forced schedule only where that schedule says top-down.  Evaluated identically by
// every CTA from state fixed before this launch.
template <typename T>
__device__ __forceinline__ bool commit_sparse(const BatchArgs<T> &a, const GroupCtrl<T> *c, int lc) {
  if (c->dir != 0 || !c->td_mark) return false;
  // every write marks at most one chunk: the level's write count bounds the marked ones
  if (a.lstat[(size_t)(c - a.ctrl) * MAXL + lc].writes * 4ull > (unsigned long long)a.nchunk32) return false;
  const uint32_t next = (uint32_t)lc + 1;
  switch (a.pol.mode) {
    case 0: case 1: return true;
    case 2: return next < a.pol.bu_from;
    default: return next - 1 < a.pol.sched_len ? a.pol.sched[next - 1] == 0 : true;
  }
}

template <typename T>
__device__ __forceinline__ void prefetch_commit_tile(const BatchArgs<T> &a, int g, int lc, size_t base) {
  const uint32_t nvt = (uint32_t)min((size_t)CTILE, (size_t)a.nva - base);
  const uint32_t wb = (nvt * (uint32_t)sizeof(T) + 15u) & ~15u, db = (nvt * 4u + 15u) & ~15u;
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(snap(a, g, lc) + base), "r"(wb) : "memory");
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a.visited + (size_t)g * a.gstride + base), "r"(wb)
               : "memory");
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a.deg + base), "r"(db) : "memory");
}

template <typename T>
__device__ __forceinline__ void commit_tile(const BatchArgs<T> &a, CommitSmem<T> &cm, int g, int lc, size_t base,
                                            unsigned long long &nf, unsigned long long &mf,
                                            unsigned long long &newp, T &nacc, bool sample,
                                            float (&bc)[WordBits<T>::value / 32], bool sparse) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  GroupCtrl<T> *c = a.ctrl + g;
  const T active = c->active;
  T *N = snap(a, g, lc);
  T *Z = snap(a, g, lc + 1);  // target of the next level's expand
  T *vis = a.visited + (size_t)g * a.gstride;
  uint32_t *qlen = c->qlen[lc & 1];
  const size_t nv = a.nva;
  T n[CVT], vv[CVT];
  uint32_t dg[CVT], rdg[CVT];  // out-degree (top-down rows), in-degree (bottom-up rows)
  bool live[CVT];              // chunk to read (dense commit, or marked dirty)
  uint8_t *dfl = a.dirty + (size_t)g * a.nchunk32;
  uint8_t fl[CVT];
#pragma unroll
  for (int k = 0; k < CVT; ++k) {
    const size_t ch = (base + (size_t)k * BLOCK + (size_t)(warp * 32)) >> 5;  // warp-uniform chunk
    fl[k] = ch < a.nchunk32 ? dfl[ch] : (uint8_t)0;
    n[k] = wzero_value<T>();
    vv[k] = wzero_value<T>();
    dg[k] = rdg[k] = 0;
  }
  if (!sparse) {  // dense: the word loads do not wait for the chunk flags
#pragma unroll
    for (int k = 0; k < CVT; ++k) {
      const size_t v = base + (size_t)k * BLOCK + tid;
      live[k] = true;
      if (v < nv) {
        n[k] = ld(N + v);
        vv[k] = ld(vis + v);
        dg[k] = __ldg(a.deg + v);
        rdg[k] = a.directed ? __ldg(a.rdeg + v) : dg[k];
      }
    }
  } else {
#pragma unroll
    for (int k = 0; k < CVT; ++k) {
      const size_t v = base + (size_t)k * BLOCK + tid;
      live[k] = fl[k] != 0;
      if (v < nv && live[k]) {
        n[k] = ld(N + v);
        vv[k] = ld(vis + v);
        dg[k] = __ldg(a.deg + v);
        rdg[k] = a.directed ? __ldg(a.rdeg + v) : dg[k];
      }
    }
  }
#pragma unroll
  for (int k = 0; k < CVT; ++k)
    if (fl[k] && lane == 0) dfl[(base + (size_t)k * BLOCK + (size_t)(warp * 32)) >> 5] = 0;  // consumed
  uint32_t bal[CVT][4];
  uint32_t wc[4] = {0, 0, 0, 0};
#pragma unroll
  for (int k = 0; k < CVT; ++k) {
    const size_t v = base + (size_t)k * BLOCK + tid;
    const bool in = v < nv;
    if (in && !a.clean_ring) st(Z + v, wzero_value<T>());
    {  // an unfiltered top-down level may have ORed already-visited bits: mask them
      const T m = wandn(n[k], vv[k]);
      if (in && !weq(m, n[k])) st(N + v, m);
      n[k] = m;
    }
    const bool nz = !wzero(n[k]);
    if (nz) st(vis + v, wor(vv[k], n[k]));
    {  // frontier bitmap of level lc + 1 (read by its bottom-up gathers); every chunk is
       // rewritten, sparse commits included (their untouched chunks hold no new bit)
      const uint32_t fball = __ballot_sync(FULL, nz);
      const size_t ch = (base + (size_t)k * BLOCK + (size_t)(warp * 32)) >> 5;
      if (lane == 0 && ch < a.nchunk32) a.fbits[(size_t)g * a.nchunk32 + ch] = fball;
    }
    if (sparse) {  // block-uniform: the new vertices of a sparse level go to the late list
      const uint32_t lb = __ballot_sync(FULL, nz);
      if (lb) {
        const int leader = __ffs(lb) - 1;
        uint32_t base0 = 0;
        if (lane == leader) base0 = atomicAdd(a.late_n + g, (uint32_t)__popc(lb));
        base0 = __shfl_sync(FULL, base0, leader);
        const uint32_t i = base0 + __popc(lb & lanemask_lt());
        if (nz && i < a.late_cap)
          a.late[(size_t)g * a.late_cap + i] = ((unsigned long long)lc << 32) | (unsigned long long)v;
      }
    }
    const T tp = (in && !sparse) ? wandn(active, wor(vv[k], n[k])) : wzero_value<T>();
    const bool un = !wzero(tp);
    const uint32_t d = dg[k], rd = rdg[k];
    if (nz) {
      nf++;
      mf += d;
      newp += wpopc(n[k]);
      nacc = wor(nacc, n[k]);
    }
    // top-down classes by out-degree, bottom-up classes by in-degree (a vertex without
    // in-edges can never be found bottom-up and is not queued)
    const bool qd = d > 0 && d <= (uint32_t)HUB_T;
    const bool light = d <= (uint32_t)LIGHT_DEG;
    const bool rqd = rd > 0 && rd <= (uint32_t)HUB_T;
    const bool rlight = rd <= (uint32_t)LIGHT_DEG;
    bal[k][Q_TDL] = __ballot_sync(FULL, nz && qd && light);
    bal[k][Q_TDH] = __ballot_sync(FULL, nz && qd && !light);
    bal[k][Q_BUL] = __ballot_sync(FULL, un && rqd && rlight);
    bal[k][Q_BUH] = __ballot_sync(FULL, un && rqd && !rlight);
    // hubs: their chunks, never the vertex queues (rare: one vote in the common case)
    if (__any_sync(FULL, in && (d > (uint32_t)HUB_T || rd > (uint32_t)HUB_T))) {
      push_hub_chunks(a, g, qlen, Q_TDC, in && nz && d > (uint32_t)HUB_T, (uint32_t)v);
      push_hub_chunks(a, g, qlen, Q_BUC, in && un && rd > (uint32_t)HUB_T, (uint32_t)v);
    }
#pragma unroll
    for (int cls = 0; cls < 4; ++cls) wc[cls] += __popc(bal[k][cls]);
  }
  if (!sparse) {  // block-uniform
    // heavy vertices (degree > SPLIT_HEAVY) enter the per-instance frontier edge counts
    // exactly on every tile, in sampled units (d / SAMPLE): a hub-dominated frontier is
    // not left to the 1/SAMPLE lottery; the light ones below are sampled
#pragma unroll
    for (int k = 0; k < CVT; ++k) {
      const bool hv = !wzero(n[k]) && dg[k] > (uint32_t)SPLIT_HEAVY;
      uint32_t hb = __ballot_sync(FULL, hv);
      while (hb) {
        const int src = __ffs(hb) - 1;
        hb &= hb - 1;
        const float dd = (float)__shfl_sync(FULL, dg[k], src) * (1.0f / (float)SAMPLE);
#pragma unroll
        for (int p = 0; p < WordBits<T>::value / 32; ++p)
          if ((__shfl_sync(FULL, wpiece(n[k], p), src) >> lane) & 1u) bc[p] += dd;
      }
    }
  }
  if (sample && !sparse) {  // block-uniform
    const uint32_t d0 = (wzero(n[0]) || dg[0] > (uint32_t)SPLIT_HEAVY) ? 0u : dg[0];
    const uint32_t dmax = __reduce_or_sync(FULL, d0);
    if (dmax) {
      const int nb = 32 - __clz(dmax);
#pragma unroll
      for (int p = 0; p < WordBits<T>::value / 32; ++p) {
        const uint32_t m = warp_transpose32(wpiece(n[0], p));
        unsigned long long sum = 0;
        for (int b = 0; b < nb; ++b) sum += (unsigned long long)__popc(m & __ballot_sync(FULL, (d0 >> b) & 1u)) << b;
        bc[p] += (float)sum;
      }
    }
  }
  if (lane == 0)
    for (int cls = 0; cls < 4; ++cls) cm.wcnt[warp][cls] = wc[cls];
  __syncthreads();
  if (tid < 4) {
    uint32_t tot = 0;
    for (int w = 0; w < NWARP; ++w) {
      const uint32_t x = cm.wcnt[w][tid];
      cm.wcnt[w][tid] = tot;  // exclusive warp offsets
      tot += x;
    }
    cm.qbase[tid] = tot ? atomicAdd(qlen + tid, tot) : 0u;
  }
  __syncthreads();
#pragma unroll
  for (int cls = 0; cls < 4; ++cls) {
    uint32_t off = cm.qbase[cls] + cm.wcnt[warp][cls];
    uint32_t *q = queue_of(a, g, cls);
#pragma unroll
    for (int k = 0; k < CVT; ++k) {
      const uint32_t b = bal[k][cls];
      if ((b >> lane) & 1u) {
        const uint32_t i = off + __popc(b & lanemask_lt());
        const uint32_t v = (uint32_t)(base + (size_t)k * BLOCK + tid);
        if (cls & 1) q[nv - 1 - i] = v; else q[i] = v;
      }
      off += __popc(b);
    }
  }
  __syncthreads();  // wcnt / qbase reused by the next tile
}

// Add one CTA's counters for group g (ntiles tiles) to the group, and if they complete the
// group's tiles, decide the next level: direction (reading #7), the per-instance split of
// a BU level (include/ibfs.h IBFS_SPLIT_*), active mask, done.
template <typename T>
__device__ void commit_flush(const BatchArgs<T> &a, CommitSmem<T> &cm, int g, int lc, uint32_t ntiles,
                             uint32_t tiles_per_group, unsigned long long nf, unsigned long long mf,
                             unsigned long long newp, T nacc, float (&bc)[WordBits<T>::value / 32],
                             bool sparse) {
  constexpr int W = WordBits<T>::value;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  GroupCtrl<T> *c = a.ctrl + g;
  if (lc >= 128 && !wzero(nacc)) atomicExch(a.range_err, 1u);  // depth > 127
  nf = warp_sum64(nf);
  mf = warp_sum64(mf);
  newp = warp_sum64(newp);
  nacc = warp_or(nacc);
  if (lane == 0) {
    cm.red[warp][0] = nf; cm.red[warp][1] = mf; cm.red[warp][2] = newp;
    cm.orr[warp] = nacc;
  }
#pragma unroll
  for (int p = 0; p < W / 32; ++p)
    if (bc[p] != 0.f) { atomicAdd(&cm.bcnt[p * 32 + lane], bc[p]); bc[p] = 0.f; }
  __syncthreads();
  if (tid < W) {
    const float x = cm.bcnt[tid];
    if (x != 0.f) atomicAdd(&c->bitw[tid], x);
    cm.bcnt[tid] = 0.f;
  }
  if (tid == 0) {
    unsigned long long t0 = 0, t1 = 0, t2 = 0;
    T o = wzero_value<T>();
    for (int k = 0; k < NWARP; ++k) {
      t0 += cm.red[k][0]; t1 += cm.red[k][1]; t2 += cm.red[k][2];
      o = wor(o, cm.orr[k]);
    }
    if (t0) atomicAdd(&c->n_f, t0);
    if (t1) atomicAdd(&c->m_f, t1);
    if (t2) atomicAdd(&c->newp, t2);
    if (!wzero(o)) red_or(&c->newacc, o);
  }
  __threadfence();
  __syncthreads();
  if (tid == 0) {
    const uint32_t prev = atomicAdd(&c->arrive, ntiles);
    cm.last = (prev + ntiles == tiles_per_group) ? 1u : 0u;
  }
  __syncthreads();
  if (!cm.last) return;  // block-uniform
  __threadfence();
  const T act = ldv(&c->newacc);
  // split: the active instances to expand top-down if the next level is BU -- Beamer's
  // rule per instance (reading #7): j stays bottom-up only while its frontier edge count
  // m_f(j) * split_div exceeds its unexplored edge count m_u(j) = ne - sum of the earlier
  // frontiers' edges (both sampled); FORCE: j % split_mod == 0
  if (tid < W / 32) cm.tdb[tid] = 0;
  if (tid == 0) cm.wmax = 0u;
  __syncthreads();
  if (a.pol.split_rel > 0.f && tid < W && ((wpiece(act, tid >> 5) >> (tid & 31)) & 1u))
    atomicMax(&cm.wmax, __float_as_uint(*(volatile float *)&c->bitw[tid]));  // w >= 0: bits order as values
  __syncthreads();
  if (tid < W) {
    const float w = *(volatile float *)&c->bitw[tid];
    const float cum = *(volatile float *)&c->cumw[tid] + w;
    c->bitw[tid] = 0.f;
    c->cumw[tid] = cum;
    bool small;
    if (a.pol.split == 2) small = (uint32_t)tid % a.pol.split_mod == 0;
    else {
      const double mf = (double)w * SAMPLE, mu = fmax((double)a.pol.ne - (double)cum * SAMPLE, 1.0);
      small = mf * (double)a.pol.split_div < mu;
      // a laggard among the group's instances keeps every bottom-up scan running to the
      // end of the row: expand it top-down too (performance only, never the result)
      if (a.pol.split_rel > 0.f && w * a.pol.split_rel < __uint_as_float(cm.wmax)) small = true;
    }
    if (a.pol.split != 1 && small && ((wpiece(act, tid >> 5) >> (tid & 31)) & 1u))
      atomicOr(&cm.tdb[tid >> 5], 1u << (tid & 31));
  }
  __syncthreads();
  if (tid == 0) {
    const unsigned long long n_f = ldv(&c->n_f), m_f = ldv(&c->m_f), np = ldv(&c->newp);
    const uint32_t cur = c->dir;
    LevelStat *ls = a.lstat + (size_t)g * MAXL + lc;
    ls->dir = cur + 1;
    ls->newp = np;
    ls->nf = n_f;
    bool bu;
    T tdb = wzero_value<T>();
    bu = !sparse && decide_bu(a.pol, (uint32_t)lc + 1, cur, n_f, m_f);
    if (bu) {
      tdb = wfrom_pieces<T>(cm.tdb);
      // auto: if every active instance is small the level is plain top-down
      if (a.pol.mode == 0 && weq(tdb, act)) { bu = false; tdb = wzero_value<T>(); }
    }
    c->active = act;
    c->newacc = wzero_value<T>();
    c->n_f = c->m_f = c->newp = 0;
    c->dir = bu ? 1u : 0u;
    c->td_bits = tdb;
    c->td_mark = (!bu && (double)m_f <= 2.0 * (double)a.nva) ? 1u : 0u;
    c->bu_probe = a.pol.bu_probe == 2 || (a.pol.bu_probe == 1 && n_f * 8ull < (unsigned long long)a.nva) ? 1u : 0u;
    // top-down pre-check of visited[w] only once a fair share of the (vertex, active
    // instance) pairs is visited; before that nearly every OR is new and the gather is
    // wasted (the commit masks what an unfiltered OR set twice)
    c->vpairs += np;
    c->td_filter = (double)c->vpairs * 2.0 > (double)a.nva * (double)wpopc(act) ? 1u : 0u;
    c->arrive = 0;
    c->sparse = sparse ? 1u : 0u;
    ls->flags = sparse ? 2u : 0u;
    if (IBFS_DEPTH_SKIP && sparse && lc < 128 && *(volatile uint32_t *)(a.late_n + g) <= a.late_cap) {
      c->skip_lv[lc >> 6] |= 1ull << (lc & 63);
      ls->flags |= 1u;
    }
    c->last_level = (uint32_t)lc;
    for (int k = 0; k < NQ; ++k) c->qlen[(lc + 1) & 1][k] = 0;  // target of commit lc+1
    if (wzero(act) || (a.pol.max_depth != 0 && (uint32_t)lc >= a.pol.max_depth)) {
      c->done = 1;
      __threadfence();
      atomicAdd(a.batch_done, 1u);
    } else if (lc + 1 < MAXL) {
      // Eq. 1 counters of level lc+1 known here: TD -- |JFQ| = vertices with new bits,
      // sum_j |FQ_j| = new pairs; BU -- the isolated vertices (never in the queues; every
      // active instance is unvisited there), the expand adds the queued ones and hubs.
      LevelStat *nx = a.lstat + (size_t)g * MAXL + lc + 1;
      if (!bu) {
        nx->jfq = n_f;
        nx->fq = np;
      } else {
        nx->jfq = a.n_iso;
        nx->fq = (unsigned long long)a.n_iso * (unsigned long long)wpopc(act);
      }
    }
  }
}

// Sparse commit with the clean ring: only the marked 32-vertex chunks can
// hold bits of S_l (every write of the level marked its chunk and the slot started at
// zero), so the warps of the whole grid scan the group's chunk map (16 flags per lane and
// step) and commit each marked chunk warp-cooperatively, lane = vertex: mask S_l with
// ~visited, visited |= S_l, the late-list entry, the top-down queue classes (no bottom-up
// queue: the next level is top-down), the counters.  The frontier bitmap is not rewritten:
// a sparse commit forces the next level top-down, only bottom-up levels read the bitmap,
// and the next dense commit rewrites it whole.  Each taking part CTA flushes once.
template <typename T>
__device__ void commit_sparse_chunks(const BatchArgs<T> &a, CommitSmem<T> &cm, int g, int lc, uint32_t rank,
                                     uint32_t K) {
  constexpr int NP = WordBits<T>::value / 32;
  const int lane = threadIdx.x & 31;
  GroupCtrl<T> *c = a.ctrl + g;
  uint32_t *qlen = c->qlen[lc & 1];
  T *N = snap(a, g, lc);
  T *vis = a.visited + (size_t)g * a.gstride;
  uint8_t *dfl = a.dirty + (size_t)g * a.nchunk32;
  unsigned long long nf = 0, mf = 0, newp = 0;
  T nacc = wzero_value<T>();
  const size_t nc = a.nchunk32;
  const size_t gw = (size_t)rank * NWARP + (threadIdx.x >> 5), nw = (size_t)K * NWARP;
  const bool al = (reinterpret_cast<uintptr_t>(dfl) & 15u) == 0;
  for (size_t c0 = gw * 512; c0 < nc; c0 += nw * 512) {  // 512 flags per warp step
    const size_t cl = c0 + (size_t)lane * 16;
    uint32_t f[4] = {0u, 0u, 0u, 0u};
    if (al && cl + 16 <= nc) {
      const uint4 x = *reinterpret_cast<const uint4 *>(dfl + cl);
      f[0] = x.x; f[1] = x.y; f[2] = x.z; f[3] = x.w;
    } else {
      for (int b = 0; b < 16; ++b)
        if (cl + b < nc && dfl[cl + b]) f[b >> 2] |= 1u << (8 * (b & 3));
    }
    uint32_t hit = 0;  // bit b: flag b of this lane's 16 is set
#pragma unroll
    for (int b = 0; b < 16; ++b) hit |= ((f[b >> 2] >> (8 * (b & 3))) & 0xffu) ? (1u << b) : 0u;
    uint32_t lanes = __ballot_sync(FULL, hit != 0);
    while (lanes) {
      const int src = __ffs(lanes) - 1;
      lanes &= lanes - 1;
      uint32_t h = __shfl_sync(FULL, hit, src);
      while (h) {
        const int b = __ffs(h) - 1;
        h &= h - 1;
        const size_t ch = c0 + (size_t)src * 16 + b;
        const size_t v = ch * 32 + lane;
        const bool in = v < a.nva;
        T n = wzero_value<T>(), vv = wzero_value<T>();
        uint32_t d = 0;
        if (in) {
          n = ld(N + v);
          vv = ld(vis + v);
          d = __ldg(a.deg + v);
        }
        const T m = wandn(n, vv);  // an unfiltered top-down OR may have set visited bits
        if (in && !weq(m, n)) st(N + v, m);
        const bool nz = !wzero(m);
        if (nz) {
          st(vis + v, wor(vv, m));
          nf++;
          mf += d;
          newp += wpopc(m);
          nacc = wor(nacc, m);
        }
        const uint32_t lb = __ballot_sync(FULL, nz);  // the late list (skipped level)
        if (lb) {
          const int leader = __ffs(lb) - 1;
          uint32_t base0 = 0;
          if (lane == leader) base0 = atomicAdd(a.late_n + g, (uint32_t)__popc(lb));
          base0 = __shfl_sync(FULL, base0, leader);
          const uint32_t i = base0 + __popc(lb & lanemask_lt());
          if (nz && i < a.late_cap)
            a.late[(size_t)g * a.late_cap + i] = ((unsigned long long)lc << 32) | (unsigned long long)v;
        }
        const bool qd = d > 0 && d <= (uint32_t)HUB_T, light = d <= (uint32_t)LIGHT_DEG;
        queue_push(a, g, qlen, Q_TDL, nz && qd && light, (uint32_t)v);
        queue_push(a, g, qlen, Q_TDH, nz && qd && !light, (uint32_t)v);
        push_hub_chunks(a, g, qlen, Q_TDC, nz && d > (uint32_t)HUB_T, (uint32_t)v);
        if (lane == 0) dfl[ch] = 0;  // consumed
      }
    }
  }
  float bc[NP];
#pragma unroll
  for (int p = 0; p < NP; ++p) bc[p] = 0.f;
  commit_flush(a, cm, g, lc, 1u, K, nf, mf, newp, nacc, bc, true);
}

// Grid-wide barrier of a cooperative launch (every CTA resident): sense-reversing, one
// counter and one generation word per batch.
__device__ __forceinline__ void grid_barrier(uint32_t *bar) {
  __syncthreads();
  if (threadIdx.x == 0) {
    volatile uint32_t *gen = bar + 1;
    const uint32_t my_gen = *gen;
    __threadfence();
    const uint32_t nb = gridDim.x * gridDim.y;
    if (atomicAdd(bar, 1u) == nb - 1) {
      bar[0] = 0;
      __threadfence();
      atomicAdd(bar + 1, 1u);
    } else {
      while (*gen == my_gen) __nanosleep(32);
    }
    __threadfence();
  }
  __syncthreads();
}

// ---------------------------------------------------------------------- level ----
// THE per-level kernel (north_star: "a single kernel per level builds the joint frontier
// queue and expands it"), one cooperative launch for all groups of a batch:
//   phase 1 (level > 1): commit of level l-1 over every (group, vertex tile) -- visited
//            |= S_l-1, zero slot l, build the JFQs of level l (Alg. 2), counters; the CTA
//            completing a group decides its direction for level l;
//   grid barrier (the expand must see committed words: Lemma C2, reading #4);
//   phase 2: expand of level l (Alg. 1) from those queues.
// Level 1's queues come from the init kernels.  A batch whose groups are all finished
// (flags final before this launch) exits at once.
template <typename T>
__global__ void __launch_bounds__(BLOCK, IBFS_EXPAND_MINB) level_kernel(BatchArgs<T> a, int level) {
  __shared__ ExpandSmem sm;
  __shared__ T s_red[NWARP];
  __shared__ CommitSmem<T> cm;
  __shared__ uint32_t s_live;
  extern __shared__ __align__(16) unsigned char dyn_smem[];
  TileQueue<T> &tq = *reinterpret_cast<TileQueue<T> *>(dyn_smem);
  const int tid = threadIdx.x;
  if (tid == 0) {
    uint32_t live = 0;
    for (int g = 0; g < a.G; ++g) live += a.ctrl[g].done ? 0u : 1u;
    s_live = live;
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    if (live) atomicMin(a.tstamp + (size_t)level * 3, t);
  }
  __syncthreads();
  if (s_live == 0) return;  // uniform: every CTA reads the same final flags
  if (level > 1) {
    const int lc = level - 1;
    const uint32_t tpg = (uint32_t)((a.nva + CTILE - 1) / CTILE);
    const size_t total = (size_t)a.G * tpg;
    int cur_g = -1;
    bool sparse = false;
    uint32_t ntiles = 0;
    unsigned long long nf = 0, mf = 0, newp = 0;
    T nacc = wzero_value<T>();
    constexpr int NP = WordBits<T>::value / 32;
    float bc[NP];
#pragma unroll
    for (int p = 0; p < NP; ++p) bc[p] = 0.f;
    for (int j = tid; j < WordBits<T>::value; j += BLOCK) cm.bcnt[j] = 0.f;
    // each group's commit kind, from state fixed before this launch: read here, before
    // this CTA arrives for any group (a group's last CTA rewrites dir / td_mark, which
    // commit_sparse reads, once every CTA has arrived for it)
    __shared__ uint8_t s_sparse[MAX_G];
    for (int g = tid; g < a.G; g += BLOCK) s_sparse[g] = (!a.ctrl[g].done && commit_sparse(a, a.ctrl + g, lc)) ? 1 : 0;
    __syncthreads();
    for (size_t w = blockIdx.x; w < total; w += gridDim.x) {
      const int g = (int)(w / tpg);
      if (g != cur_g) {
        if (cur_g >= 0 && ntiles) commit_flush(a, cm, cur_g, lc, ntiles, tpg, nf, mf, newp, nacc, bc, sparse);
        cur_g = g;
        sparse = s_sparse[g] != 0;
        ntiles = 0;
        nf = mf = newp = 0;
        nacc = wzero_value<T>();
      }
      if (a.ctrl[g].done) continue;  // finished before this launch (stable)
      const uint32_t tix = (uint32_t)(w % tpg);
      if (sparse && a.clean_ring) continue;  // the chunk scan below commits it
      if (tid == 0 && !sparse) {
        // the commit streams S_l, visited and the degrees of its tiles: ask the TMA unit to
        // prefetch this group's tile two tiles (of this CTA) ahead into L2
        // (cp.async.bulk.prefetch.L2), so its loads hit L2 instead of waiting on DRAM
        const size_t tn = (size_t)tix + 2 * (size_t)gridDim.x;
        if (tn < tpg) prefetch_commit_tile(a, g, lc, tn * CTILE);
      }
      commit_tile(a, cm, g, lc, (size_t)tix * CTILE, nf, mf, newp, nacc, tix % SAMPLE_TILES == 0, bc, sparse);
      ++ntiles;
    }
    if (cur_g >= 0 && ntiles) commit_flush(a, cm, cur_g, lc, ntiles, tpg, nf, mf, newp, nacc, bc, sparse);
    if (a.clean_ring) {
      const uint32_t K = min(gridDim.x, max(1u, (uint32_t)((a.nchunk32 + NWARP * 2048 - 1) / (NWARP * 2048))));
      for (int g = 0; g < a.G; ++g) {
        if (!s_sparse[g]) continue;
        const uint32_t rank = (blockIdx.x + gridDim.x - (uint32_t)(((size_t)g * K) % gridDim.x)) % gridDim.x;
        if (rank < K) commit_sparse_chunks(a, cm, g, lc, rank, K);
      }
    }
    grid_barrier(a.gbar);
  }
  if (tid == 0 && blockIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    a.tstamp[(size_t)level * 3 + 1] = t;
  }
  expand_phase(a, level, sm, s_red, tq);
  __syncthreads();
  if (tid == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    atomicMax(a.tstamp + (size_t)level * 3 + 2, t);
  }
}

// ------------------------------------------------------------------------ depth ----
// Depth rows from the level snapshots l in [l0, l1] (l1 capped at the group's last
// committed level and at 127): depth[j][v] = the first l with bit j of S_l[v] set.
//
// A CTA works through tiles of DV = 128 consecutive caller-id vertices (columns) x all W
// rows.  The tile's vertices of degree > 0 are one contiguous range [c0, c0 + k) of
// compacted ids, so each level's words for the tile are one contiguous run: a producer
// warp fetches them with 1-D TMA bulk copies (cp.async.bulk, up to DLB levels per stage,
// DNS stages on mbarriers), DNS - 1 tiles ahead of the consumers.
//   phase A (accumulate): the k words of a level are dealt densely -- consumer thread t
//     owns dense slot t % 64 (+ 64 in a second round when k > 64) for the W/4 instances
//     of part t / 64, so no lane idles on an isolated column -- and accumulates (l + 1)
//     into the byte of every instance whose bit first appears at level l (SIMD within a
//     register: bytes never carry, each receives at most one value <= 128).  The column
//     bytes go to a column-major staging tile in shared memory (16-byte chunks, XOR
//     swizzled by column).
//   phase B (store): thread t takes column t % 128 in caller order for the W/2
//     instances of half t / 128 (isolated columns: all -1), turns l + 1 into l (0 -> -1),
//     and a 4 x 4 byte transpose among the 4 lanes of consecutive columns (2 shuffles + 2
//     byte permutes per word) gives each lane 4 consecutive columns of one row: a warp
//     stores 4 rows x 32 contiguous bytes per instruction (full 32-byte sectors,
//     streaming stores -- the rows are written once and not re-read here).
// first != 0 writes every byte; otherwise (a ring-slot flush before reuse) only the bytes
// found in [l0, l1] change.  m_s and the isolated sources' own zero are separate passes.
constexpr int DV = 128;               // columns per tile
constexpr int DCW = 8;                // consumer warps
constexpr int DTHREADS = DCW * 32;    // consumer threads
constexpr int DSLOTS = 64;            // dense slots per round (DTHREADS / 4 parts)
#ifndef IBFS_DEPTH_DLB
#define IBFS_DEPTH_DLB 5
#endif
#ifndef IBFS_DEPTH_MINB
#define IBFS_DEPTH_MINB 3
#endif
constexpr int DLB = IBFS_DEPTH_DLB;   // levels per pipeline stage
constexpr int DNS = 3;                // pipeline stages
constexpr int DHDR = 32 + DV;         // stage header: k, run offset, c0, read mask, nzbits[4]; slot -> column table

__device__ __forceinline__ uint32_t spread4(uint32_t nib) {
  // 4-bit nibble -> 0x01 in each byte whose bit is set
  return (nib * 0x00204081u) & 0x01010101u;
}

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(unsigned long long *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(unsigned long long *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long *bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// Wait for phase `parity` to complete; the thread is suspended inside try_wait (time
// hint) instead of spinning on the issue slots.
__device__ __forceinline__ void mbar_wait(unsigned long long *bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
      " @!p bra WAIT_%=;\n}\n" ::"r"(smem_u32(bar)),
      "r"(parity), "r"(1000000u)
      : "memory");
}
// 1-D TMA bulk copy global -> shared (16-byte aligned, size a multiple of 16), completing
// `bytes` of transaction count on the mbarrier.
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, unsigned long long *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// barrier among the DTHREADS consumer threads only (the producer warp never joins)
__device__ __forceinline__ void consumers_sync() { asm volatile("bar.sync 1, %0;" ::"n"(DTHREADS) : "memory"); }

// explicit shared-space accesses (32-bit shared addresses)
__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds16(uint32_t a) {
  unsigned short v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint32_t lds8(uint32_t a) {
  unsigned short v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=h"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint4 lds128(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) { asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v)); }
__device__ __forceinline__ void sts64(uint32_t a, uint32_t x, uint32_t y) {
  asm volatile("st.shared.v2.u32 [%0], {%1,%2};" ::"r"(a), "r"(x), "r"(y));
}
__device__ __forceinline__ void sts128(uint32_t a, uint32_t x, uint32_t y, uint32_t z, uint32_t w) {
  asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(a), "r"(x), "r"(y), "r"(z), "r"(w));
}

// the W/4-bit part p of a status word at shared address a (little-endian pieces)
template <int PB>
__device__ __forceinline__ uint32_t lds_part(uint32_t a) {
  if (PB == 32) return lds32(a);
  if (PB == 16) return lds16(a);
  return lds8(a);
}

template <typename T>
struct DepthLayout {
  static constexpr int W = WordBits<T>::value;
  static constexpr size_t COLB = (size_t)DV * W;                     // one column-major staging tile
  static constexpr size_t SROW = (size_t)DV * sizeof(T) + 16;        // one level's run (+ slack)
  static constexpr size_t STAGE = DHDR + DLB * SROW;
  static constexpr size_t BYTES = 128 + 2 * COLB + DNS * STAGE;      // + 128 for alignment
  static_assert(DHDR % 16 == 0 && SROW % 16 == 0 && STAGE % 16 == 0, "stage runs must stay 16-byte aligned");
};

template <typename T>
constexpr size_t depth_smem_bytes() {
  return DepthLayout<T>::BYTES;
}

// byte offset of chunk `ch` (16 bytes) of column `col` in a column-major staging tile
template <int W>
__device__ __forceinline__ uint32_t colb_off(uint32_t col, uint32_t ch) {
  constexpr uint32_t NCH = W / 16;  // chunks per column
  return col * (uint32_t)W + ((ch ^ (col & (NCH - 1))) << 4);
}

// Warp roles: warps 0 .. DCW - 1 consume; warp DCW produces (all lanes write the header's
// dense slot -> column table, lane 0 issues the copies).  Stage st is "full" when the 32
// producer lanes arrived and its bytes landed (s_full[st], one expect_tx), "empty" when
// every consumer warp has read it (s_empty[st]).
template <typename T>
__global__ void __launch_bounds__(DTHREADS + 32, IBFS_DEPTH_MINB)
    depth_kernel(BatchArgs<T> a, int l0, int l1, int first) {
  using L = DepthLayout<T>;
  constexpr int W = WordBits<T>::value;
  constexpr int PB = W / 4;        // instances per part (phase A)
  constexpr int PQ = PB / 4;       // byte registers per part
  constexpr int HW = W / 8;        // byte registers per half column (phase B)
  constexpr int NCH = W / 16;      // 16-byte chunks per column
  extern __shared__ unsigned char dsm_raw[];
  const uint32_t sbase = (smem_u32(dsm_raw) + 127u) & ~127u;
  const uint32_t colb = sbase;                   // [2][DV][W] column-major staging
  const uint32_t stage_base = sbase + 2 * (uint32_t)L::COLB;
  __shared__ __align__(8) unsigned long long s_full[DNS], s_empty[DNS];
  const int g = blockIdx.y;
  const int rows = group_rows(a, g);
  if (rows == 0) return;
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  const GroupCtrl<T> *c = a.ctrl + g;
  const int last = min((int)c->last_level, min(l1, 127));
  const int nlev = last - l0 + 1;  // levels to read (may be <= 0)
  const unsigned long long sk0 = c->skip_lv[0], sk1 = c->skip_lv[1];
  auto skipped = [&](int l) { return ((l < 64 ? sk0 >> l : sk1 >> (l - 64)) & 1ull) != 0; };
  if (nlev <= 0 && !first) return;
  const int nbat = nlev > 0 ? (nlev + DLB - 1) / DLB : 1;  // >= 1 job per tile (its header)
  const size_t nvv = a.nv;
  const size_t ntiles = (nvv + DV - 1) / DV;
  const size_t my_tiles = blockIdx.x < ntiles ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  const size_t njobs = my_tiles * (size_t)nbat;
  if (t == 0) {
    for (int k = 0; k < DNS; ++k) {
      mbar_init(&s_full[k], 32);
      mbar_init(&s_empty[k], DCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == DCW) {
    // ---- producer: job jb = (tile jb / nbat of this CTA, batch jb % nbat) -> stage jb % DNS
    for (size_t jb = 0; jb < njobs; ++jb) {
      const int st = (int)(jb % DNS);
      const int b = (int)(jb % nbat);
      const size_t tix = blockIdx.x + (jb / nbat) * gridDim.x;
      const uint32_t c0 = __ldg(a.tbase + tix), k = __ldg(a.tbase + tix + 1) - c0;
      const uint4 nzw = __ldg(reinterpret_cast<const uint4 *>(a.nzbits) + tix);  // bits beyond nv are 0
      const int lb = l0 + b * DLB, le = min(last, lb + DLB - 1);
      const int nl = le >= lb ? le - lb + 1 : 0;
      uint32_t off = 0, size = 0;
      if (k && nl) {
        const uintptr_t src0 = (uintptr_t)(snap(a, g, lb) + c0);
        off = (uint32_t)(src0 & 15u);
        size = (uint32_t)((off + (size_t)k * sizeof(T) + 15) & ~(size_t)15);
      }
      if (jb >= (size_t)DNS) mbar_wait(&s_empty[st], (uint32_t)((jb / DNS - 1) & 1));
      const uint32_t sb = stage_base + (uint32_t)(st * L::STAGE);
      // dense slot -> column table: lane l places the columns 4l .. 4l + 3 of degree > 0
      const uint32_t wv = lane < 8 ? nzw.x : lane < 16 ? nzw.y : lane < 24 ? nzw.z : nzw.w;
      const uint32_t nib = (wv >> (4 * (lane & 7))) & 0xFu;
      const uint32_t cnt = __popc(nib);
      uint32_t incl = cnt;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(FULL, incl, d);
        if (lane >= d) incl += y;
      }
      uint32_t pos = incl - cnt;
#pragma unroll
      for (int cc = 0; cc < 4; ++cc)
        if ((nib >> cc) & 1u) {
          asm volatile("st.shared.u8 [%0], %1;" ::"r"(sb + 32 + pos), "h"((unsigned short)(4 * lane + cc)));
          ++pos;
        }
      uint32_t rmask = 0;  // bit u: level lb + u is in range and its snapshot is loaded
      for (int l = lb; l <= le; ++l) rmask |= skipped(l) ? 0u : 1u << (l - lb);
      if (lane == 0) {
        sts128(sb, k, off, c0, rmask);
        sts128(sb + 16, nzw.x, nzw.y, nzw.z, nzw.w);
      }
      const uint32_t total = size * (uint32_t)__popc(rmask);
      if (lane == 0) mbar_arrive_expect_tx(&s_full[st], total); else mbar_arrive(&s_full[st]);
      if (lane == 0)
        for (int l = lb; l <= le && total; ++l) {
          if (!((rmask >> (l - lb)) & 1u)) continue;
          const unsigned char *src = reinterpret_cast<const unsigned char *>(snap(a, g, l) + c0) - off;
          bulk_g2s(sb + DHDR + (uint32_t)((l - lb) * L::SROW), src, size, &s_full[st]);
        }
    }
  } else {
    // ---- consumers
    const int part = t / DSLOTS, dslot = t % DSLOTS;      // phase A
    const int col = t % DV, half = t / DV;                // phase B
    const int q4 = lane & 3;                               // lane within its column quad
    const uint32_t sel1 = (q4 & 1) ? 0x3726u : 0x5140u;
    const uint32_t sel2 = (q4 & 2) ? 0x3276u : 0x5410u;
    const int rowperm = (q4 == 1) ? 2 : (q4 == 2 ? 1 : q4);  // row held after the transpose
    const bool word_ok = (nvv % 4) == 0;
    size_t job = 0;
    int buf = 0;
    for (size_t tix = blockIdx.x; tix < ntiles; tix += gridDim.x, buf ^= 1) {
      const size_t v0 = tix * DV;
      const uint32_t cb = colb + (uint32_t)(buf * L::COLB);
      uint32_t acc[2][PQ];
#pragma unroll
      for (int r = 0; r < 2; ++r)
#pragma unroll
        for (int q = 0; q < PQ; ++q) acc[r][q] = 0;
      uint32_t reached[2] = {0u, 0u};
      uint32_t k = 0, mynz = 0, dcol[2] = {0u, 0u};
      for (int b = 0; b < nbat; ++b, ++job) {
        const int st = (int)(job % DNS);
        mbar_wait(&s_full[st], (uint32_t)((job / DNS) & 1));
        const uint32_t sb = stage_base + (uint32_t)(st * L::STAGE);
        const uint32_t off = lds32(sb + 4), rm = lds32(sb + 12);  // rm: header's read mask
        if (b == 0) {
          k = lds32(sb);
          mynz = (lds32(sb + 16 + 4 * (col >> 5)) >> (col & 31)) & 1u;
#pragma unroll
          for (int r = 0; r < 2; ++r) {
            const uint32_t i = (uint32_t)(dslot + DSLOTS * r);
            if (i < k) dcol[r] = lds8(sb + 32 + i);
          }
        }
        const int lb = l0 + b * DLB;
#pragma unroll
        for (int r = 0; r < 2; ++r) {
          const uint32_t i = (uint32_t)(dslot + DSLOTS * r);
          if (i < k) {
            const uint32_t p = sb + DHDR + off + i * (uint32_t)sizeof(T) + (uint32_t)(part * PB / 8);
#pragma unroll
            for (int u = 0; u < DLB; ++u) {
              // out of range, or not loaded (late_fix_kernel writes those depths)
              if (!((rm >> u) & 1u)) continue;
              const uint32_t hb = lds_part<PB>(p + (uint32_t)(u * L::SROW)) & ~reached[r];
              if (!hb) continue;
              const uint32_t inc = (uint32_t)(lb + u + 1);
              if (reached[r] == 0u && hb == (PB == 32 ? 0xffffffffu : ((1u << PB) - 1u))) {
                // the whole part at one level (common): no bit spreading
#pragma unroll
                for (int q = 0; q < PQ; ++q) acc[r][q] = inc * 0x01010101u;
              } else {
#pragma unroll
                for (int q = 0; q < PQ; ++q) acc[r][q] += spread4((hb >> (4 * q)) & 0xFu) * inc;
              }
              reached[r] |= hb;
            }
          }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&s_empty[st]);  // this warp is done with stage st
      }
      // phase A -> staging (dense slot i of the tile is column dcol, from the stage table)
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        const uint32_t i = (uint32_t)(dslot + DSLOTS * r);
        if (i < k) {
          const uint32_t dc = dcol[r];
          const uint32_t byte0 = (uint32_t)(part * PB);  // first instance of the part
          if (PB == 32) {
            sts128(cb + colb_off<W>(dc, byte0 / 16), acc[r][0], acc[r][1], acc[r][2], acc[r][3]);
            sts128(cb + colb_off<W>(dc, byte0 / 16 + 1), acc[r][4 % PQ], acc[r][5 % PQ], acc[r][6 % PQ],
                   acc[r][7 % PQ]);
          } else if (PB == 16) {
            sts128(cb + colb_off<W>(dc, byte0 / 16), acc[r][0], acc[r][1 % PQ], acc[r][2 % PQ], acc[r][3 % PQ]);
          } else {
            sts64(cb + colb_off<W>(dc, byte0 / 16) + (byte0 & 15u), acc[r][0], acc[r][1 % PQ]);
          }
        }
      }
      consumers_sync();  // staging complete (and the previous tile's readers of this buffer are done)
      // phase B: column `col`, rows half * W/2 .. + W/2 - 1
      uint32_t x[HW];
      if (mynz) {
#pragma unroll
        for (int cq = 0; cq < HW / 4; ++cq) {
          const uint4 v = lds128(cb + colb_off<W>((uint32_t)col, (uint32_t)(half * (NCH / 2) + cq)));
          x[4 * cq] = v.x; x[4 * cq + 1] = v.y; x[4 * cq + 2] = v.z; x[4 * cq + 3] = v.w;
        }
      } else {
#pragma unroll
        for (int q = 0; q < HW; ++q) x[q] = 0;
      }
      const size_t cbase = v0 + (size_t)(col & ~3);  // first column of this lane's quad
      const int row0 = half * (W / 2) + rowperm;
      int8_t *dst = a.out + ((size_t)g * W + row0) * nvv + cbase;  // row row0 + 4q at dst + 4q nv
      const bool fast = word_ok && v0 + DV <= nvv && first && rows == W;  // block-uniform
#pragma unroll
      for (int q = 0; q < HW; ++q, dst += 4 * nvv) {
        uint32_t w = __vsub4(x[q], 0x01010101u);  // l + 1 -> l, 0 -> 0xff (-1)
        uint32_t y = __shfl_xor_sync(FULL, w, 1);
        w = __byte_perm(w, y, sel1);
        y = __shfl_xor_sync(FULL, w, 2);
        w = __byte_perm(w, y, sel2);
        if (fast) {
          __stcs(reinterpret_cast<unsigned int *>(dst), w);
        } else {
          if (row0 + 4 * q >= rows) continue;
          const uint32_t ff = __vcmpeq4(w, 0xffffffffu);
          if (word_ok && v0 + DV <= nvv && ff == 0) {
            __stcs(reinterpret_cast<unsigned int *>(dst), w);
          } else {
#pragma unroll
            for (int bb = 0; bb < 4; ++bb)
              if (cbase + bb < nvv && (first || !((ff >> (8 * bb)) & 1u))) dst[bb] = (int8_t)(w >> (8 * bb));
          }
        }
      }
    }
  }
}

// ---- depth rows, TMA-store variant (the default when the rows allow it) ----
// The store pattern decides this kernel's speed: 4-byte streaming stores that put 32 bytes
// in each of 4 rows per warp instruction top out at ~1.7 TB/s on B200 (profiles/r02/
// randbench.json "st32_rows_gbs"; every 32-byte sector is its own L2 write request), while
// whole 128-byte lines stream at ~6.2 TB/s.  So the rows of a 128-column x W-row tile are
// assembled row-major in shared memory and leave as ONE 2-D bulk tensor store (TMA,
// cp.async.bulk.tensor): full lines, no store instructions on the SM, no lane transposes.
//   fill    the tile's buffer = 0xff (-1: isolated columns, unreached instances);
//   phase A as in depth_kernel (thread = dense slot x instance part, SIMD-within-register
//           accumulation of l + 1 over the loaded snapshot levels), then each thread writes
//           its column's bytes straight into their rows (byte stores; a warp = 32 columns
//           of one row: one shared-memory wavefront);
//   store   fence.proxy.async, barrier, one thread issues the tensor store; the buffer is
//           reused two tiles later, after cp.async.bulk.wait_group.read.
// Only for a batch's first (complete) flush; ring-slot re-flushes and rows that break the
// tensor map's alignment rules use depth_kernel.
#ifndef IBFS_DTMA_DLB
#define IBFS_DTMA_DLB 5
#endif
#ifndef IBFS_DTMA_NS
#define IBFS_DTMA_NS 4
#endif
#ifndef IBFS_DTMA_MINB
#define IBFS_DTMA_MINB 3
#endif
constexpr int DLB2 = IBFS_DTMA_DLB;  // loaded snapshot levels per pipeline stage
constexpr int DNS2 = IBFS_DTMA_NS;   // pipeline stages
constexpr int DMAXL = 128;           // levels a flush can cover (depths <= 127)

template <typename T>
struct DepthTmaLayout {
  static constexpr int W = WordBits<T>::value;
  static constexpr size_t TILE = (size_t)DV * W;                     // one row-major output tile
  static constexpr size_t SROW = (size_t)DV * sizeof(T) + 16;
  static constexpr size_t STAGE = DHDR + DLB2 * SROW;
  static constexpr size_t BYTES = 128 + 2 * TILE + DNS2 * STAGE;
  static_assert(TILE % 128 == 0 && STAGE % 16 == 0, "tiles stay 128-byte aligned");
  static_assert(DLB2 <= 16, "stage header holds 16 level bytes");
};

template <typename T>
constexpr size_t depth_tma_smem_bytes() {
  return DepthTmaLayout<T>::BYTES;
}

__device__ __forceinline__ void sts8(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "r"(v));
}

// Stage header (DHDR bytes): [0] k (non-isolated columns of the tile), [4] byte offset of
// the runs, [8] c0, [12] nl (loaded levels in this stage), [16 .. 16 + DLB2) the level + 1 of
// each slot, [32 .. 32 + DV) dense slot -> column.  A tile takes ceil(loaded levels / DLB2)
// stages (at least one, for its header); only loaded levels occupy slots.
template <typename T>
__global__ void __launch_bounds__(DTHREADS + 32, IBFS_DTMA_MINB)
    depth_tma_kernel(const __grid_constant__ CUtensorMap tmap, BatchArgs<T> a, int l0, int l1, int zero_runs) {
  using L = DepthTmaLayout<T>;
  constexpr int W = WordBits<T>::value;
  constexpr int PB = W / 4;   // instances per part
  constexpr int PQ = PB / 4;  // byte registers per part
  extern __shared__ unsigned char dsm_raw[];
  const uint32_t sbase = (smem_u32(dsm_raw) + 127u) & ~127u;
  const uint32_t outb = sbase;  // [2][W][DV] row-major output tiles
  const uint32_t stage_base = sbase + 2 * (uint32_t)L::TILE;
  // clean ring, fused (W = 128: one 16-byte word per vertex): once the consumers have read
  // a stage, its snapshot runs have landed in shared memory, so they overwrite the runs in
  // global memory with zeros (one streaming store per vertex and loaded level, spread over
  // the consumer threads) and the ring is zero again without a separate pass
  const bool zr = zero_runs != 0 && sizeof(T) == 16;
  __shared__ __align__(8) unsigned long long s_full[DNS2], s_empty[DNS2];
  __shared__ const T *s_run[DMAXL];  // snapshot array of each loaded level, in level order
  __shared__ uint8_t s_inc[DMAXL];   // its level + 1
  __shared__ int s_nload;
  const int g = blockIdx.y;
  const int rows = group_rows(a, g);
  if (rows == 0) return;
  const int t = threadIdx.x, lane = t & 31, warp = t >> 5;
  const GroupCtrl<T> *c = a.ctrl + g;
  const int last = min((int)c->last_level, min(l1, 127));
  const size_t nvv = a.nv;
  const size_t ntiles = (nvv + DV - 1) / DV;
  if (t == 0) {
    // the loaded levels (skipped ones come from the late list / source list): their ring
    // slot arrays, computed once
    const unsigned long long sk0 = c->skip_lv[0], sk1 = c->skip_lv[1];
    int n = 0;
    for (int l = l0; l <= last; ++l) {
      const bool sk = ((l < 64 ? sk0 >> l : sk1 >> (l - 64)) & 1ull) != 0;
      if (sk) continue;
      s_run[n] = snap(a, g, l);
      s_inc[n] = (uint8_t)(l + 1);
      ++n;
    }
    s_nload = n;
    for (int k = 0; k < DNS2; ++k) {
      mbar_init(&s_full[k], 32);
      mbar_init(&s_empty[k], DCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int nload = s_nload;
  const int nbat = nload > 0 ? (nload + DLB2 - 1) / DLB2 : 1;  // >= 1 stage per tile (its header)
  const size_t my_tiles = blockIdx.x < ntiles ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  const size_t njobs = my_tiles * (size_t)nbat;
  const uint32_t full0 = smem_u32(&s_full[0]), empty0 = smem_u32(&s_empty[0]);
  if (warp == DCW) {
    // ---- producer: job jb = (tile jb / nbat of this CTA, stage batch jb % nbat)
    int st = 0;
    uint32_t ph = 0;
    for (size_t jb = 0; jb < njobs; ++jb) {
      const int b = (int)(jb % nbat);
      const size_t tix = blockIdx.x + (jb / nbat) * gridDim.x;
      const uint32_t c0 = __ldg(a.tbase + tix), k = __ldg(a.tbase + tix + 1) - c0;
      const int s0 = b * DLB2, nl = max(0, min(DLB2, nload - s0));
      uint32_t off = 0, size = 0;
      if (k && nl) {
        const uintptr_t src0 = (uintptr_t)(s_run[s0] + c0);
        off = (uint32_t)(src0 & 15u);
        size = (uint32_t)((off + (size_t)k * sizeof(T) + 15) & ~(size_t)15);
      }
      if (jb >= (size_t)DNS2) mbar_wait(reinterpret_cast<unsigned long long *>(&s_empty[st]), ph ^ 1u);
      const uint32_t sb = stage_base + (uint32_t)(st * L::STAGE);
      if (b == 0) {  // the tile's dense slot -> column table (read by the consumers at b == 0)
        const uint4 nzw = __ldg(reinterpret_cast<const uint4 *>(a.nzbits) + tix);
        const uint32_t wv = lane < 8 ? nzw.x : lane < 16 ? nzw.y : lane < 24 ? nzw.z : nzw.w;
        const uint32_t nib = (wv >> (4 * (lane & 7))) & 0xFu;
        const uint32_t cnt = __popc(nib);
        uint32_t incl = cnt;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const uint32_t y = __shfl_up_sync(FULL, incl, d);
          if (lane >= d) incl += y;
        }
        uint32_t pos = incl - cnt;
#pragma unroll
        for (int cc = 0; cc < 4; ++cc)
          if ((nib >> cc) & 1u) {
            asm volatile("st.shared.u8 [%0], %1;" ::"r"(sb + 32 + pos), "h"((unsigned short)(4 * lane + cc)));
            ++pos;
          }
      }
      if (lane < nl) sts8(sb + 16 + lane, s_inc[s0 + lane]);
      if (lane == 0) sts128(sb, k, off, c0, (uint32_t)nl);
      const uint32_t total = size * (uint32_t)nl;
      if (lane == 0) mbar_arrive_expect_tx(&s_full[st], total); else mbar_arrive(&s_full[st]);
      if (lane < nl && total) {
        const unsigned char *src = reinterpret_cast<const unsigned char *>(s_run[s0 + lane] + c0) - off;
        bulk_g2s(sb + DHDR + (uint32_t)(lane * L::SROW), src, size, &s_full[st]);
      }
      if (++st == DNS2) { st = 0; ph ^= 1u; }
    }
  } else {
    // ---- consumers
    const int part = t / DSLOTS, dslot = t % DSLOTS;
    int st = 0;
    uint32_t ph = 0;
    int buf = 0;
    for (size_t tix = blockIdx.x; tix < ntiles; tix += gridDim.x, buf ^= 1) {
      const uint32_t ob = outb + (uint32_t)(buf * L::TILE);
      // the tensor store issued from this buffer two tiles ago has finished reading it
      if (t == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      consumers_sync();
#pragma unroll
      for (uint32_t j = 0; j < (uint32_t)(L::TILE / 16 / DTHREADS); ++j)
        sts128(ob + 16 * ((uint32_t)t + j * DTHREADS), 0xffffffffu, 0xffffffffu, 0xffffffffu, 0xffffffffu);
      uint32_t acc[2][PQ];
#pragma unroll
      for (int r = 0; r < 2; ++r)
#pragma unroll
        for (int q = 0; q < PQ; ++q) acc[r][q] = 0;
      uint32_t reached[2] = {0u, 0u};
      uint32_t k = 0, dcol[2] = {0u, 0u};
      for (int b = 0; b < nbat; ++b) {
        asm volatile(
            "{\n .reg .pred p;\n WAIT_%=:\n"
            " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
            " @!p bra WAIT_%=;\n}\n" ::"r"(full0 + 8u * (uint32_t)st),
            "r"(ph), "r"(1000000u)
            : "memory");
        const uint32_t sb = stage_base + (uint32_t)(st * L::STAGE);
        const uint4 hdr = lds128(sb);  // k, off, c0, nl
        if (b == 0) {
          k = hdr.x;
#pragma unroll
          for (int r = 0; r < 2; ++r) {
            const uint32_t i = (uint32_t)(dslot + DSLOTS * r);
            if (i < k) dcol[r] = lds8(sb + 32 + i);
          }
        }
        const uint32_t nl = hdr.w;
        const uint4 incs = lds128(sb + 16);
#pragma unroll
        for (int r = 0; r < 2; ++r) {
          const uint32_t i = (uint32_t)(dslot + DSLOTS * r);
          if (i < k) {
            const uint32_t p = sb + DHDR + hdr.y + i * (uint32_t)sizeof(T) + (uint32_t)(part * PB / 8);
#pragma unroll
            for (int u = 0; u < DLB2; ++u) {
              if ((uint32_t)u >= nl) break;
              const uint32_t hb = lds_part<PB>(p + (uint32_t)(u * L::SROW)) & ~reached[r];
              if (!hb) continue;
              const uint32_t iw = u < 4 ? incs.x : u < 8 ? incs.y : u < 12 ? incs.z : incs.w;
              const uint32_t inc = (iw >> (8 * (u & 3))) & 0xffu;
              if (reached[r] == 0u && hb == (PB == 32 ? 0xffffffffu : ((1u << PB) - 1u))) {
#pragma unroll
                for (int q = 0; q < PQ; ++q) acc[r][q] = inc * 0x01010101u;
              } else if (PB == 32) {
                // byte b of word q holds instance q + 8b (not 4q + b): its bit is (hb >> q)
                // bit 8b, so the spread is one shift and one mask
#pragma unroll
                for (int q = 0; q < PQ; ++q) acc[r][q] += ((hb >> q) & 0x01010101u) * inc;
              } else {
#pragma unroll
                for (int q = 0; q < PQ; ++q) acc[r][q] += spread4((hb >> (4 * q)) & 0xFu) * inc;
              }
              reached[r] |= hb;
            }
          }
        }
        if (zr) {  // the stage's runs are in shared memory: zero them in the ring
          for (uint32_t u = 0; u < nl; ++u) {
            uint4 *dst = reinterpret_cast<uint4 *>(const_cast<T *>(s_run[b * DLB2 + (int)u]) + hdr.z);
            for (uint32_t i = (uint32_t)t; i < k; i += DTHREADS) __stcs(dst + i, make_uint4(0u, 0u, 0u, 0u));
          }
        }
        __syncwarp();
        if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(empty0 + 8u * (uint32_t)st) : "memory");
        if (++st == DNS2) { st = 0; ph ^= 1u; }
      }
      consumers_sync();  // the 0xff fill is complete
      // the column's bytes into their rows (a warp writes 32 columns of one row per store):
      // byte bb of word q is instance q + 8 bb (W = 128) or 4q + bb (W = 32, 64) of the part
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        const uint32_t i = (uint32_t)(dslot + DSLOTS * r);
        if (i < k) {
          const uint32_t base = ob + (uint32_t)(part * PB) * DV + dcol[r];
#pragma unroll
          for (int q = 0; q < PQ; ++q) {
            const uint32_t w = __vsub4(acc[r][q], 0x01010101u);  // l + 1 -> l, 0 -> 0xff (-1)
#pragma unroll
            for (int bb = 0; bb < 4; ++bb) {
              const uint32_t inst = PB == 32 ? (uint32_t)(q + 8 * bb) : (uint32_t)(4 * q + bb);
              sts8(base + inst * DV, w >> (8 * bb));
            }
          }
        }
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      consumers_sync();
      if (t == 0) {
        const int c0i = (int)(tix * DV), r0i = g * W;
        asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                         reinterpret_cast<uint64_t>(&tmap)),
                     "r"(ob), "r"(c0i), "r"(r0i)
                     : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    }
    if (t == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  }
}

// --------------------------------------------------------------------- finalize ----
// m_s (reading #11): m_s[j] = sum_v deg(v) * bit j of visited[v] over
// the final visited words (compacted ids: isolated vertices have degree 0).  A warp takes
// 32 vertices at a time: a 32 x 32 bit transpose per 32-bit piece gives lane i the mask
// M of the warp's vertices reached by instance 32p + i, and the degree-weighted count is
// sum_b popc(M & D_b) << b over the degree bit planes D_b = ballot(bit b of deg).
template <typename T>
__global__ void __launch_bounds__(BLOCK) ms_kernel(BatchArgs<T> a, unsigned long long *m_out, int zl0, int zl1) {
  constexpr int W = WordBits<T>::value;
  constexpr int NP = W / 32;
  __shared__ unsigned long long s_m[W];
  __shared__ T *s_zero[DMAXL];  // clean ring: the loaded snapshot slots this pass zeroes
  __shared__ int s_nz;
  const int g = blockIdx.y;
  const int rows = group_rows(a, g);
  // a group finished at init (every source isolated) never zeroed its visited words; its
  // instances reach nothing of positive degree: m_s = 0
  if (rows == 0 || a.ctrl[g].last_level == 0xffffffffu) return;
  const int tid = threadIdx.x, lane = tid & 31;
  for (int j = tid; j < W; j += BLOCK) s_m[j] = 0;
  if (tid == 0) {
    // zl0 <= zl1: also return the loaded slots of levels [zl0, zl1] to zero (the clean
    // ring's pass fused into this ALU-bound one: the stores overlap the bit transposes)
    const GroupCtrl<T> *c = a.ctrl + g;
    const int last = min((int)c->last_level, min(zl1, 127));
    const unsigned long long sk0 = c->skip_lv[0], sk1 = c->skip_lv[1];
    int n = 0;
    for (int l = zl0; l <= last && n < DMAXL; ++l)
      if (((l < 64 ? sk0 >> l : sk1 >> (l - 64)) & 1ull) == 0) s_zero[n++] = snap(a, g, l);
    s_nz = n;
  }
  __syncthreads();
  const int nzs = s_nz;
  const T *vis = a.visited + (size_t)g * a.gstride;
  unsigned long long acc[NP];
  uint32_t cnt[NP][8];  // popcounts per (piece, degree bit plane < 8), weighted at the end
#pragma unroll
  for (int p = 0; p < NP; ++p) {
    acc[p] = 0;
#pragma unroll
    for (int b = 0; b < 8; ++b) cnt[p][b] = 0;
  }
  const size_t nvr = ((size_t)a.nva + 31) & ~(size_t)31;  // warp-uniform trip count
  for (size_t v = (size_t)blockIdx.x * BLOCK + tid; v < nvr; v += (size_t)gridDim.x * BLOCK) {
    const bool in = v < a.nva;
    // coherent load: with the clean ring this thread zeroes the word below (the
    // non-coherent path could be ordered after that store)
    const T x = in ? ld(vis + v) : wzero_value<T>();
    const uint32_t d = in ? __ldg(a.deg + v) : 0u;
    if (a.clean_ring && in && !wzero(x)) st(const_cast<T *>(vis) + v, wzero_value<T>());  // visited back to zero
    if (in)
      for (int z = 0; z < nzs; ++z) st_cs(s_zero[z] + v, wzero_value<T>());
    const uint32_t any = __ballot_sync(FULL, !wzero(x) && d != 0);
    if (!any) continue;
    uint32_t m[NP];
#pragma unroll
    for (int p = 0; p < NP; ++p) m[p] = warp_transpose32(wpiece(x, p));
    // degrees < 256 through their 8 bit planes; the few larger ones (hubs) one by one
    const bool heavy = d >= 256u;
    const uint32_t dl = heavy ? 0u : d;
#pragma unroll
    for (int b = 0; b < 8; ++b) {
      const uint32_t db = __ballot_sync(FULL, (dl >> b) & 1u);
#pragma unroll
      for (int p = 0; p < NP; ++p) cnt[p][b] += __popc(m[p] & db);
    }
    uint32_t hv = __ballot_sync(FULL, heavy && !wzero(x));
    while (hv) {
      const int src = __ffs(hv) - 1;
      hv &= hv - 1;
      const unsigned long long dd = __shfl_sync(FULL, d, src);
#pragma unroll
      for (int p = 0; p < NP; ++p)
        if ((__shfl_sync(FULL, wpiece(x, p), src) >> lane) & 1u) acc[p] += dd;
    }
  }
#pragma unroll
  for (int p = 0; p < NP; ++p) {
#pragma unroll
    for (int b = 0; b < 8; ++b) acc[p] += (unsigned long long)cnt[p][b] << b;
    if (acc[p]) atomicAdd(&s_m[p * 32 + lane], acc[p]);
  }
  __syncthreads();
  for (int j = tid; j < rows; j += BLOCK)
    if (s_m[j]) atomicAdd(&m_out[(size_t)g * W + j], s_m[j]);
}

// Instances whose source is isolated (degree 0) never enter the status words: depth 0 at
// their own source, after the rows' first flush wrote -1 there.
template <typename T>
__global__ void iso_fix_kernel(BatchArgs<T> a) {
  constexpr int W = WordBits<T>::value;
  const int g = blockIdx.x;
  const int rows = group_rows(a, g);
  for (int j = threadIdx.x; j < rows; j += blockDim.x)
    if (a.csrc[(size_t)g * W + j] == NO_VERTEX)
      a.out[((size_t)g * W + j) * a.nv + a.src[(size_t)g * W + j]] = 0;
}

// Depths of the levels the depth kernel skipped (GroupCtrl::skip_lv), in [l0, l1]:
// level 0 from the source list, the sparse-committed levels from the late list -- each
// entry (l, v) writes l into the byte of every instance whose bit is in S_l[v].  Runs
// after depth_kernel of the same flush (its first pass wrote -1 there).
__device__ __forceinline__ uint32_t caller_id(const uint32_t *tbase, const uint32_t *nzbits, uint32_t ntiles,
                                              uint32_t v) {
  uint32_t lo = 0, hi = ntiles;  // last 128-column tile with tbase <= v
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(tbase + mid) <= v) lo = mid; else hi = mid;
  }
  uint32_t r = v - __ldg(tbase + lo);
  for (uint32_t w = 4 * lo;; ++w) {
    const uint32_t m = __ldg(nzbits + w), c = __popc(m);
    if (r < c) return 32 * w + __fns(m, 0, (int)r + 1);
    r -= c;
  }
}

template <typename T>
__global__ void late_fix_kernel(BatchArgs<T> a, int l0, int l1) {
  constexpr int W = WordBits<T>::value;
  const int g = blockIdx.y;
  const int rows = group_rows(a, g);
  if (rows == 0) return;
  const GroupCtrl<T> *c = a.ctrl + g;
  if (c->last_level == 0xffffffffu) return;  // done at init: nothing was traversed
  const int last = min((int)c->last_level, min(l1, 127));
  const unsigned long long sk0 = c->skip_lv[0], sk1 = c->skip_lv[1];
  auto skipped = [&](int l) { return ((l < 64 ? sk0 >> l : sk1 >> (l - 64)) & 1ull) != 0; };
  const size_t nvv = a.nv;
  if (l0 == 0 && skipped(0) && blockIdx.x == 0)
    for (int j = threadIdx.x; j < rows; j += blockDim.x)
      if (a.csrc[(size_t)g * W + j] != NO_VERTEX) {
        a.out[((size_t)g * W + j) * nvv + a.src[(size_t)g * W + j]] = 0;
        // S_0 holds bits only at the sources (duplicates store the same zero)
        if (a.clean_ring) st(snap(a, g, 0) + a.csrc[(size_t)g * W + j], wzero_value<T>());
      }
  const uint32_t n = min(a.late_n[g], a.late_cap);
  const uint32_t ntiles = (uint32_t)((nvv + 127) / 128);
  for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < n; e += gridDim.x * blockDim.x) {
    const unsigned long long ent = a.late[(size_t)g * a.late_cap + e];
    const int l = (int)(ent >> 32);
    const uint32_t v = (uint32_t)ent;
    if (l < l0 || l > last || !skipped(l)) continue;
    // a coherent load: the non-coherent path (ldg) may be scheduled after the clean-ring
    // store below, which would read the zero
    T *sp = snap(a, g, l) + v;
    const T x = ld(sp);
    const size_t col = caller_id(a.tbase, a.nzbits, ntiles, v);
#pragma unroll
    for (int p = 0; p < W / 32; ++p) {
      uint32_t m = wpiece(x, p);
      while (m) {
        const int j = 32 * p + __ffs(m) - 1;
        m &= m - 1;
        if (j < rows) a.out[((size_t)g * W + j) * nvv + col] = (int8_t)l;
      }
    }
    if (a.clean_ring) st(sp, wzero_value<T>());  // the one entry per (level, vertex)
  }
}

// Clean ring (BatchArgs::clean_ring): after the depth rows of levels [l0, l1] are written,
// zero the snapshot slots the depth kernel read (every level <= last_level that was not
// skipped) with 16-byte streaming stores; the skipped levels' few entries were zeroed by
// late_fix_kernel.  Levels past a group's last_level were never written (the expand of a
// finished group does not run).  The ring is then all zero again for the next batch, so the
// commits need not clear the slot of the next level (16 B per vertex and level, sparse
// tail levels included).
template <typename T>
__global__ void __launch_bounds__(BLOCK) ring_clean_kernel(BatchArgs<T> a, int l0, int l1) {
  const int g = blockIdx.y;
  if (group_rows(a, g) == 0) return;
  const GroupCtrl<T> *c = a.ctrl + g;
  if (c->last_level == 0xffffffffu) return;
  const int last = min((int)c->last_level, min(l1, 127));
  const unsigned long long sk0 = c->skip_lv[0], sk1 = c->skip_lv[1];
  const size_t n16 = (size_t)a.nva * sizeof(T) / 16 + 1;  // slot words rounded up (gstride pads)
  const size_t stride = (size_t)gridDim.x * BLOCK;
  const uint4 z = make_uint4(0u, 0u, 0u, 0u);
  for (int l = l0; l <= last; ++l) {
    if (((l < 64 ? sk0 >> l : sk1 >> (l - 64)) & 1ull) != 0) continue;
    uint4 *p = reinterpret_cast<uint4 *>(snap(a, g, l));
    for (size_t i = (size_t)blockIdx.x * BLOCK + threadIdx.x; i < n16; i += stride) __stcs(p + i, z);
  }
}

// IBFS_CHECK_RING (tests): flag = 1 if any of the n16 16-byte words is non-zero.
__global__ void ring_check_kernel(const uint4 *p, size_t n16, uint32_t *flag) {
  uint32_t acc = 0;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x) {
    const uint4 x = p[i];
    acc |= x.x | x.y | x.z | x.w;
  }
  if (__syncthreads_or(acc != 0) && threadIdx.x == 0) atomicExch(flag, 1u);
}

__device__ __forceinline__ unsigned long long splitmix64(unsigned long long z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// digest[r] = sum over v with depth >= 0 of splitmix64((v << 8) | (depth + 1)).
template <typename T>
__global__ void __launch_bounds__(BLOCK) digest_kernel(BatchArgs<T> a, unsigned long long *d_out) {
  constexpr int W = WordBits<T>::value;
  const int r = blockIdx.y;  // row within the batch
  const int g = r / W, j = r % W;
  if (j >= group_rows(a, g)) return;
  const int8_t *row = a.out + (size_t)r * a.nv;
  unsigned long long s = 0;
  for (size_t v = (size_t)blockIdx.x * BLOCK + threadIdx.x; v < a.nv; v += (size_t)gridDim.x * BLOCK) {
    const int d = row[v];
    if (d >= 0) s += splitmix64(((unsigned long long)v << 8) | (unsigned long long)(d + 1));
  }
  s = warp_sum64(s);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(&d_out[r], s);
}

}  // namespace ibfs
