// kernels.cuh -- the per-level kernels of the joint bitwise traversal (sm_100a).
//
// One group = up to W BFS instances sharing one W-bit status word per vertex (the
// Bitwise Status Array, §6).  Per group the device holds
//   visited[v]  bit j = 1 iff instance j reached v at an earlier level  (BSA_k)
//   buf0/buf1   alternate by level parity: F = discoveries of level l-1 (the top-down
//               frontier words, Alg. 2 "BSA_k+1 XOR BSA_k" P:L793), N = discoveries of
//               level l being accumulated (the new bits of BSA_k+1, Alg. 1).
// Level l (discovers depth l; reading #20) is two launches:
//   expand_kernel<T>(l): builds the joint frontier queue per vertex tile with a warp
//       ballot (Alg. 2; JFQ P:L329-L335) and expands it --
//       top-down  N[w] |= F[f] & ~visited[w]   with RED.OR (Alg. 1 l.5),
//       bottom-up acc  |= visited[w] & T[f], T = ~visited[f] & active, early exit when
//                 acc == T (Alg. 1 l.7-10; reading #5), N[f] = acc.
//   commit_kernel<T>(l): visited |= N, depth[j][v] = l for every new bit j (P:L779
//       "the differences between BSA_k and BSA_k+1 are used to identify the just visited
//       vertices"), clears the old frontier buffer, counts the direction-switch inputs,
//       and its last CTA per group decides the next level's direction (reading #7).
// Work decomposition (static, built at load): edge-balanced vertex tiles of at most
// V_TILE vertices / E_TILE non-hub edges, plus hub chunks of CHUNK edges for vertices of
// degree > HUB_T (the paper's shared-memory "cache" of a frontier's adjacency shared by
// all instances, becomes a CTA-cooperative expansion of the hub's row).
#pragma once
#include <cstdint>
#include "word.cuh"

namespace ibfs {

constexpr int BLOCK = 256;
constexpr int NWARP = BLOCK / 32;
constexpr int V_TILE = 1024;
constexpr int E_TILE = 8192;
constexpr int HUB_T = 8192;
constexpr int CHUNK = 8192;
constexpr int BU_WARP_DEG = 32;
constexpr int MAXL = 130;       // level index 1..129 (129 only detects depth > 127)
constexpr int MAX_G = 64;       // groups per launch batch
constexpr unsigned FULL = 0xffffffffu;

struct HubChunk {
  unsigned long long e0, e1;
  uint32_t v;
  uint32_t first;
};

// Per group per level counters (device).  dir: 0 = level not run, 1 = TD, 2 = BU.
struct LevelStat {
  unsigned long long jfq, fq, proc, insp, writes, newp, nf;
  uint32_t dir, pad;
};

template <typename T>
struct GroupCtrl {
  T active;   // instances that discovered something at the last committed level
  T newacc;   // OR of the new bits of the running commit
  unsigned long long n_f, m_f, m_u, newp;
  uint32_t dir;     // direction of the next expand: 0 TD, 1 BU
  uint32_t done;
  uint32_t arrive;
  uint32_t last_level;
};

struct Policy {
  uint32_t mode;      // IBFS_DIR_*
  uint32_t bu_from;
  float alpha, beta;
  unsigned long long nv_active;  // vertices with degree > 0
  uint32_t sched_len;
  uint8_t sched[MAXL];  // 0 TD / 1 BU for level l at index l-1
};

template <typename T>
struct BatchArgs {
  const unsigned long long *off;
  const uint32_t *adj;
  const uint32_t *deg;
  uint32_t nv;
  size_t gstride;  // words per per-group array
  T *visited, *buf0, *buf1;
  GroupCtrl<T> *ctrl;
  LevelStat *lstat;     // [G][MAXL]
  uint32_t *work_ctr;   // [MAXL]
  uint32_t *batch_done;
  uint32_t *range_err;
  int G;
  uint32_t n_total;     // sources in the whole run
  uint32_t group0;      // global index of this batch's first group
  const uint32_t *src;  // this batch's sources, group-major, row g*W + j
  int8_t *out;          // row g*W + j of this batch at out + (g*W + j) * nv
  const HubChunk *chunks;
  uint32_t n_chunks;
  const uint32_t *tile_begin;  // [n_tiles + 1]
  uint32_t n_tiles;
  Policy pol;
};

template <typename T>
__device__ __forceinline__ int group_rows(const BatchArgs<T> &a, int g) {
  constexpr int W = WordBits<T>::value;
  long long r = (long long)a.n_total - (long long)(a.group0 + g) * W;
  return r >= W ? W : (r > 0 ? (int)r : 0);
}

template <typename T>
__device__ __forceinline__ T *frontier_buf(const BatchArgs<T> &a, int g, int level) {
  return ((level - 1) & 1 ? a.buf1 : a.buf0) + (size_t)g * a.gstride;
}
template <typename T>
__device__ __forceinline__ T *next_buf(const BatchArgs<T> &a, int g, int level) {
  return (level & 1 ? a.buf1 : a.buf0) + (size_t)g * a.gstride;
}

__device__ __forceinline__ uint32_t lanemask_lt() {
  uint32_t m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// ------------------------------------------------------------------------- init ----
// Zero the group's status arrays and fill its depth rows with -1 (a2).
template <typename T>
__global__ void __launch_bounds__(BLOCK) init_state_kernel(BatchArgs<T> a) {
  constexpr int W = WordBits<T>::value;
  const int g = blockIdx.y;
  const size_t stride = (size_t)gridDim.x * BLOCK;
  const T z = wzero_value<T>();
  T *vis = a.visited + (size_t)g * a.gstride;
  T *b0 = a.buf0 + (size_t)g * a.gstride;
  T *b1 = a.buf1 + (size_t)g * a.gstride;
  for (size_t v = (size_t)blockIdx.x * BLOCK + threadIdx.x; v < a.nv; v += stride) {
    st(vis + v, z);
    st(b0 + v, z);
    st(b1 + v, z);
  }
  const int rows = group_rows(a, g);
  if (rows == 0) return;
  int8_t *base = a.out + (size_t)g * W * a.nv;
  const size_t bytes = (size_t)rows * a.nv;
  // head bytes up to 16-byte alignment, then 16-byte stores, then the tail
  size_t head = (16 - ((uintptr_t)base & 15)) & 15;
  if (head > bytes) head = bytes;
  const size_t gid = (size_t)blockIdx.x * BLOCK + threadIdx.x;
  if (gid < head) base[gid] = -1;
  const size_t nvec = (bytes - head) / 16;
  int4 *vp = reinterpret_cast<int4 *>(base + head);
  const int4 m1 = make_int4(-1, -1, -1, -1);
  for (size_t i = gid; i < nvec; i += stride) vp[i] = m1;
  const size_t tail0 = head + nvec * 16;
  if (gid < bytes - tail0) base[tail0 + gid] = -1;
}

// Sources: visited[s_j] |= bit j, F[s_j] |= bit j, depth[j][s_j] = 0; control words.
template <typename T>
__global__ void init_sources_kernel(BatchArgs<T> a, uint32_t first_dir) {
  constexpr int W = WordBits<T>::value;
  const int g = blockIdx.x;
  const int rows = group_rows(a, g);
  T *vis = a.visited + (size_t)g * a.gstride;
  T *f = a.buf0 + (size_t)g * a.gstride;  // frontier buffer of level 1
  for (int j = threadIdx.x; j < rows; j += blockDim.x) {
    uint32_t s = a.src[(size_t)g * W + j];
    set_bit_atomic(vis + s, j);
    set_bit_atomic(f + s, j);
    a.out[((size_t)g * W + j) * a.nv + s] = 0;
  }
  LevelStat *ls = a.lstat + (size_t)g * MAXL;
  for (int l = threadIdx.x; l < MAXL; l += blockDim.x) ls[l] = LevelStat{};
  if (threadIdx.x == 0) {
    GroupCtrl<T> c;
    c.active = wlowmask<T>(rows);
    c.newacc = wzero_value<T>();
    c.n_f = c.m_f = c.m_u = c.newp = 0;
    c.dir = first_dir;
    c.done = rows == 0 ? 1u : 0u;
    c.arrive = 0;
    c.last_level = 0;
    a.ctrl[g] = c;
    if (rows == 0) atomicAdd(a.batch_done, 1u);
  }
  if (g == 0) {
    for (int l = threadIdx.x; l < MAXL; l += blockDim.x) a.work_ctr[l] = 0;
  }
}

// ----------------------------------------------------------------------- expand ----
struct ExpandSmem {
  unsigned long long start[V_TILE];
  uint32_t aux[V_TILE + 1];  // TD: degree prefix; BU: degree
  uint32_t vtx[V_TILE];
  uint32_t wsum[NWARP];
  uint32_t cnt[2];
  uint32_t item;
  uint32_t flag;
  unsigned long long acc[MAX_G][5];  // jfq, fq, proc, insp, writes
};

// Exclusive scan of s[0..n) in place (n <= V_TILE), s[n] = total.  Block-wide.
__device__ __forceinline__ void block_exclusive_scan(uint32_t *s, uint32_t n, uint32_t *wsum) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int PER = V_TILE / BLOCK;  // 4 consecutive entries per thread
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

// Largest q in [0, n) with s[q] <= e (s strictly increasing, s[0] = 0, s[n] > e).
__device__ __forceinline__ uint32_t lbs_search(const uint32_t *s, uint32_t n, uint32_t e) {
  uint32_t lo = 0, hi = n;
  while (hi - lo > 1) {
    uint32_t mid = (lo + hi) >> 1;
    if (s[mid] <= e) lo = mid; else hi = mid;
  }
  return lo;
}

template <typename T>
__device__ __forceinline__ void flush_counts(ExpandSmem &sm, int g, uint32_t jfq, uint32_t fq,
                                             uint32_t proc, uint32_t insp, uint32_t writes) {
  jfq = __reduce_add_sync(FULL, jfq);
  fq = __reduce_add_sync(FULL, fq);
  proc = __reduce_add_sync(FULL, proc);
  insp = __reduce_add_sync(FULL, insp);
  writes = __reduce_add_sync(FULL, writes);
  if ((threadIdx.x & 31) == 0) {
    if (jfq) atomicAdd(&sm.acc[g][0], (unsigned long long)jfq);
    if (fq) atomicAdd(&sm.acc[g][1], (unsigned long long)fq);
    if (proc) atomicAdd(&sm.acc[g][2], (unsigned long long)proc);
    if (insp) atomicAdd(&sm.acc[g][3], (unsigned long long)insp);
    if (writes) atomicAdd(&sm.acc[g][4], (unsigned long long)writes);
  }
}

// Top-down tile: ballot-compact the frontiers (F != 0) of the tile into a CTA-local
// JFQ, then an edge-balanced sweep over their rows (load-balanced search on the degree
// prefix), OR-ing the frontier word into each unvisited neighbour (Alg. 1 l.4-5).
template <typename T>
__device__ void tile_td(const BatchArgs<T> &a, ExpandSmem &sm, T *s_word, int g, uint32_t t,
                        int level) {
  const int tid = threadIdx.x, lane = tid & 31;
  const uint32_t vb = a.tile_begin[t], ve = a.tile_begin[t + 1];
  const T *F = frontier_buf(a, g, level);
  T *N = next_buf(a, g, level);
  const T *vis = a.visited + (size_t)g * a.gstride;
  uint32_t jfq = 0, fq = 0, insp = 0, writes = 0;
  if (tid == 0) sm.cnt[0] = 0;
  __syncthreads();
  for (uint32_t base = vb; base < ve; base += BLOCK) {
    const uint32_t v = base + tid;
    const bool in = v < ve;
    T f = in ? ldg(F + v) : wzero_value<T>();
    const bool nz = !wzero(f);
    uint32_t d = nz ? __ldg(a.deg + v) : 0u;
    const bool isq = nz && d <= (uint32_t)HUB_T;
    if (isq) { jfq++; fq += wpopc(f); }
    const bool keep = isq && d > 0;
    const uint32_t bal = __ballot_sync(FULL, keep);
    if (bal) {
      uint32_t wb = 0;
      if (lane == 0) wb = atomicAdd(&sm.cnt[0], (uint32_t)__popc(bal));
      wb = __shfl_sync(FULL, wb, 0);
      if (keep) {
        const uint32_t pos = wb + __popc(bal & lanemask_lt());
        sm.start[pos] = __ldg(a.off + v);
        s_word[pos] = f;
        sm.aux[pos] = d;
      }
    }
  }
  __syncthreads();
  const uint32_t qn = sm.cnt[0];
  block_exclusive_scan(sm.aux, qn, sm.wsum);
  const uint32_t total = sm.aux[qn];
  constexpr int U = 4;
  for (uint32_t e0 = 0; e0 < total; e0 += BLOCK * U) {
    uint32_t w[U];
    T fw[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint32_t e = e0 + u * BLOCK + tid;
      w[u] = 0xffffffffu;
      if (e < total) {
        const uint32_t q = lbs_search(sm.aux, qn, e);
        w[u] = __ldg(a.adj + sm.start[q] + (e - sm.aux[q]));
        fw[u] = s_word[q];
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (w[u] != 0xffffffffu) {
        insp++;
        const T b = wandn(fw[u], ldg(vis + w[u]));
        if (!wzero(b)) { red_or(N + w[u], b); writes++; }
      }
    }
  }
  flush_counts<T>(sm, g, jfq, fq, qn > 0 && tid == 0 ? qn : 0u, insp, writes);
}

// Bottom-up tile: every vertex with an unvisited active bit (T = ~visited & active) is a
// frontier (Alg. 2 l.7, reading #6); it ORs its neighbours' visited words masked by T,
// in CSR order, and stops as soon as the accumulated word covers T (early termination,
// P:L817 with the active mask of reading #5).  Degree <= 32: one thread per vertex;
// larger: one warp per vertex with a warp OR-reduce and a warp-wide exit test.
template <typename T>
__device__ void tile_bu(const BatchArgs<T> &a, ExpandSmem &sm, T *s_word, int g, uint32_t t,
                        int level, T active) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const uint32_t vb = a.tile_begin[t], ve = a.tile_begin[t + 1];
  T *N = next_buf(a, g, level);
  const T *vis = a.visited + (size_t)g * a.gstride;
  uint32_t jfq = 0, fq = 0, proc = 0, insp = 0, writes = 0;
  if (tid == 0) { sm.cnt[0] = 0; sm.cnt[1] = 0; }
  __syncthreads();
  for (uint32_t base = vb; base < ve; base += BLOCK) {
    const uint32_t v = base + tid;
    const bool in = v < ve;
    T tg = wzero_value<T>();
    if (in) tg = wandn(active, ldg(vis + v));
    const bool nz = !wzero(tg);
    const uint32_t d = nz ? __ldg(a.deg + v) : 0u;
    const bool isq = nz && d <= (uint32_t)HUB_T;
    if (isq) { jfq++; fq += wpopc(tg); }
    const bool small = isq && d > 0 && d <= (uint32_t)BU_WARP_DEG;
    const bool large = isq && d > (uint32_t)BU_WARP_DEG;
    const uint32_t bs = __ballot_sync(FULL, small);
    const uint32_t bl = __ballot_sync(FULL, large);
    uint32_t ws = 0, wl = 0;
    if (lane == 0) {
      if (bs) ws = atomicAdd(&sm.cnt[0], (uint32_t)__popc(bs));
      if (bl) wl = atomicAdd(&sm.cnt[1], (uint32_t)__popc(bl));
    }
    ws = __shfl_sync(FULL, ws, 0);
    wl = __shfl_sync(FULL, wl, 0);
    if (small || large) {
      const uint32_t pos = small ? ws + __popc(bs & lanemask_lt())
                                 : (uint32_t)(V_TILE - 1) - (wl + __popc(bl & lanemask_lt()));
      sm.start[pos] = __ldg(a.off + v);
      s_word[pos] = tg;
      sm.aux[pos] = d;
      sm.vtx[pos] = v;
    }
  }
  __syncthreads();
  const uint32_t ns = sm.cnt[0], nl = sm.cnt[1];
  // thread per low-degree vertex
  for (uint32_t q = tid; q < ns; q += BLOCK) {
    const unsigned long long s0 = sm.start[q];
    const uint32_t d = sm.aux[q];
    const T tg = s_word[q];
    T acc = wzero_value<T>();
    proc++;
    for (uint32_t k = 0; k < d; k += 4) {
      uint32_t w[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) w[u] = (k + u < d) ? __ldg(a.adj + s0 + k + u) : 0xffffffffu;
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (w[u] != 0xffffffffu) { acc = wor(acc, wand(ldg(vis + w[u]), tg)); insp++; }
      if (weq(acc, tg)) break;
    }
    if (!wzero(acc)) { st(N + sm.vtx[q], acc); writes++; }
  }
  // warp per higher-degree vertex
  for (uint32_t q = warp; q < nl; q += NWARP) {
    const uint32_t idx = V_TILE - 1 - q;
    const unsigned long long s0 = sm.start[idx];
    const uint32_t d = sm.aux[idx];
    const T tg = s_word[idx];
    T acc = wzero_value<T>();
    if (lane == 0) proc++;
    for (uint32_t k = 0; k < d; k += 32) {
      T x = wzero_value<T>();
      if (k + lane < d) {
        const uint32_t w = __ldg(a.adj + s0 + k + lane);
        x = wand(ldg(vis + w), tg);
        insp++;
      }
      acc = wor(acc, warp_or(x));
      if (weq(acc, tg)) break;
    }
    if (lane == 0 && !wzero(acc)) { st(N + sm.vtx[idx], acc); writes++; }
  }
  flush_counts<T>(sm, g, jfq, fq, proc, insp, writes);
}

// Hub chunk, top-down: CHUNK edges of one hub's row swept by the whole CTA.
template <typename T>
__device__ void hub_td(const BatchArgs<T> &a, ExpandSmem &sm, int g, const HubChunk c, int level) {
  const int tid = threadIdx.x;
  const T *F = frontier_buf(a, g, level);
  T *N = next_buf(a, g, level);
  const T *vis = a.visited + (size_t)g * a.gstride;
  const T f = ldg(F + c.v);
  if (wzero(f)) return;
  uint32_t insp = 0, writes = 0;
  constexpr int U = 4;
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
        const T b = wandn(f, ldg(vis + w[u]));
        if (!wzero(b)) { red_or(N + w[u], b); writes++; }
      }
    }
  }
  const bool first = c.first && tid == 0;
  flush_counts<T>(sm, g, first ? 1u : 0u, first ? (uint32_t)wpopc(f) : 0u, first ? 1u : 0u, insp,
                  writes);
}

// Hub chunk, bottom-up: the CTA ORs a chunk of the hub's neighbours in waves, with a
// block OR-reduce and an exit test per wave against T and the bits other chunks have
// already found (atomically accumulated in N[hub]).
template <typename T>
__device__ void hub_bu(const BatchArgs<T> &a, ExpandSmem &sm, T *s_red, int g, const HubChunk c,
                       int level, T active) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  T *N = next_buf(a, g, level);
  const T *vis = a.visited + (size_t)g * a.gstride;
  const T tg = wandn(active, ldg(vis + c.v));
  if (wzero(tg)) return;
  const bool first = c.first && tid == 0;
  if (tid == 0) sm.flag = weq(wand(ldv(N + c.v), tg), tg) ? 1u : 0u;
  __syncthreads();
  uint32_t insp = 0, writes = 0;
  T acc = wzero_value<T>();
  if (!sm.flag) {
    constexpr int U = 4;
    for (unsigned long long e0 = c.e0; e0 < c.e1; e0 += BLOCK * U) {
      T x = wzero_value<T>();
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const unsigned long long e = e0 + u * BLOCK + tid;
        if (e < c.e1) {
          const uint32_t w = __ldg(a.adj + e);
          x = wor(x, wand(ldg(vis + w), tg));
          insp++;
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
  flush_counts<T>(sm, g, first ? 1u : 0u, first ? (uint32_t)wpopc(tg) : 0u, first ? 1u : 0u, insp,
                  writes);
}

// One launch per level for all groups of a batch.  CTAs pull work items (hub chunks
// first, then tiles) from a per-level counter; each item carries its group, whose
// direction for this level was decided by the previous commit.
template <typename T>
__global__ void __launch_bounds__(BLOCK) expand_kernel(BatchArgs<T> a, int level) {
  __shared__ ExpandSmem sm;
  __shared__ T s_word[V_TILE];
  __shared__ T s_red[NWARP];
  const int tid = threadIdx.x;
  if (*(volatile uint32_t *)a.batch_done >= (uint32_t)a.G) return;
  for (int i = tid; i < a.G * 5; i += BLOCK) sm.acc[i / 5][i % 5] = 0ull;
  const uint32_t per_group = a.n_chunks + a.n_tiles;
  const uint32_t total = per_group * (uint32_t)a.G;
  for (;;) {
    __syncthreads();
    if (tid == 0) sm.item = atomicAdd(a.work_ctr + level, 1u);
    __syncthreads();
    const uint32_t item = sm.item;
    if (item >= total) break;
    const int g = (int)(item % (uint32_t)a.G);
    const uint32_t k = item / (uint32_t)a.G;
    const GroupCtrl<T> *c = a.ctrl + g;
    if (c->done) continue;
    const uint32_t dir = c->dir;
    if (k < a.n_chunks) {
      const HubChunk hc = a.chunks[k];
      if (dir == 0) hub_td<T>(a, sm, g, hc, level);
      else hub_bu<T>(a, sm, s_red, g, hc, level, c->active);
    } else if (dir == 0) {
      tile_td<T>(a, sm, s_word, g, k - a.n_chunks, level);
    } else {
      tile_bu<T>(a, sm, s_word, g, k - a.n_chunks, level, c->active);
    }
  }
  __syncthreads();
  for (int i = tid; i < a.G; i += BLOCK) {
    LevelStat *ls = a.lstat + (size_t)i * MAXL + level;
    if (sm.acc[i][0]) atomicAdd(&ls->jfq, sm.acc[i][0]);
    if (sm.acc[i][1]) atomicAdd(&ls->fq, sm.acc[i][1]);
    if (sm.acc[i][2]) atomicAdd(&ls->proc, sm.acc[i][2]);
    if (sm.acc[i][3]) atomicAdd(&ls->insp, sm.acc[i][3]);
    if (sm.acc[i][4]) atomicAdd(&ls->writes, sm.acc[i][4]);
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

template <typename T>
__device__ __forceinline__ bool decide_bu(const Policy &p, uint32_t next_level, uint32_t cur_dir,
                                          unsigned long long n_f, unsigned long long m_f,
                                          unsigned long long m_u) {
  if (p.mode == 1) return false;
  if (p.mode == 2) return next_level >= p.bu_from;
  if (p.mode == 3 && next_level - 1 < p.sched_len) return p.sched[next_level - 1] != 0;
  // auto (reading #7): TD -> BU when the frontier's edges m_f exceed the
  // unexplored edges m_u / alpha; BU -> TD when the frontier holds < nv_active / beta
  // vertices.
  if (cur_dir == 0) return (double)m_f * (double)p.alpha > (double)m_u && m_f > 0;
  return !((double)n_f * (double)p.beta < (double)p.nv_active);
}

template <typename T>
__global__ void __launch_bounds__(BLOCK) commit_kernel(BatchArgs<T> a, int level) {
  constexpr int W = WordBits<T>::value;
  constexpr int PIECES = W / 32;
  __shared__ unsigned long long s_red[NWARP][4];
  __shared__ T s_or[NWARP];
  __shared__ uint32_t s_last;
  const int g = blockIdx.y;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  GroupCtrl<T> *c = a.ctrl + g;
  if (*(volatile uint32_t *)&c->done) return;
  const T active = c->active;
  const T *N = next_buf(a, g, level);
  T *F = frontier_buf(a, g, level);
  T *vis = a.visited + (size_t)g * a.gstride;
  int8_t *out = a.out + (size_t)g * W * a.nv;
  const size_t nv = a.nv;
  unsigned long long nf = 0, mf = 0, mu = 0, newp = 0;
  T nacc = wzero_value<T>();
  bool range = false;
  const size_t stride = (size_t)gridDim.x * BLOCK;
  for (size_t base = (size_t)blockIdx.x * BLOCK; base < nv; base += stride) {
    const size_t v = base + tid;
    const bool in = v < nv;
    T n = wzero_value<T>();
    T vv = wzero_value<T>();
    if (in) {
      n = ld(N + v);
      vv = ld(vis + v);
      st(F + v, wzero_value<T>());
    }
    const bool nz = !wzero(n);
    if (nz) st(vis + v, wor(vv, n));
    const T tnew = in ? wandn(active, wor(vv, n)) : wzero_value<T>();
    const bool un = !wzero(tnew);
    const uint32_t d = (nz || un) ? __ldg(a.deg + v) : 0u;
    if (nz) { nf++; mf += d; newp += wpopc(n); nacc = wor(nacc, n); }
    if (un) mu += d;
    if (level <= 127) {
      // depth record: iterate the bits set anywhere in the warp so that lanes holding
      // the same instance j store to consecutive bytes of row j together
#pragma unroll
      for (int k = 0; k < PIECES; ++k) {
        const uint32_t p = wpiece(n, k);
        uint32_t any = __reduce_or_sync(FULL, p);
        while (any) {
          const int j = __ffs(any) - 1;
          any &= any - 1;
          if ((p >> j) & 1u) out[(size_t)(k * 32 + j) * nv + v] = (int8_t)level;
        }
      }
    } else if (nz) {
      range = true;
    }
  }
  if (range) atomicExch(a.range_err, 1u);
  nf = warp_sum64(nf);
  mf = warp_sum64(mf);
  mu = warp_sum64(mu);
  newp = warp_sum64(newp);
  nacc = warp_or(nacc);
  if (lane == 0) {
    s_red[warp][0] = nf; s_red[warp][1] = mf; s_red[warp][2] = mu; s_red[warp][3] = newp;
    s_or[warp] = nacc;
  }
  __syncthreads();
  if (tid == 0) {
    unsigned long long t0 = 0, t1 = 0, t2 = 0, t3 = 0;
    T o = wzero_value<T>();
    for (int k = 0; k < NWARP; ++k) {
      t0 += s_red[k][0]; t1 += s_red[k][1]; t2 += s_red[k][2]; t3 += s_red[k][3];
      o = wor(o, s_or[k]);
    }
    if (t0) atomicAdd(&c->n_f, t0);
    if (t1) atomicAdd(&c->m_f, t1);
    if (t2) atomicAdd(&c->m_u, t2);
    if (t3) atomicAdd(&c->newp, t3);
    if (!wzero(o)) red_or(&c->newacc, o);
    __threadfence();
    const uint32_t prev = atomicAdd(&c->arrive, 1u);
    s_last = (prev == gridDim.x - 1) ? 1u : 0u;
  }
  __syncthreads();
  if (s_last && tid == 0) {
    __threadfence();
    const T act = ldv(&c->newacc);
    const unsigned long long n_f = ldv(&c->n_f), m_f = ldv(&c->m_f), m_u = ldv(&c->m_u),
                             np = ldv(&c->newp);
    const uint32_t cur = c->dir;
    LevelStat *ls = a.lstat + (size_t)g * MAXL + level;
    ls->dir = cur + 1;
    ls->newp = np;
    ls->nf = n_f;
    const bool bu = decide_bu<T>(a.pol, (uint32_t)level + 1, cur, n_f, m_f, m_u);
    c->active = act;
    c->newacc = wzero_value<T>();
    c->n_f = c->m_f = c->m_u = c->newp = 0;
    c->dir = bu ? 1u : 0u;
    c->arrive = 0;
    c->last_level = (uint32_t)level;
    if (wzero(act)) {
      c->done = 1;
      __threadfence();
      atomicAdd(a.batch_done, 1u);
    }
  }
}

// --------------------------------------------------------------------- finalize ----
// m_s = sum over reached v of deg(v) (reading #11), from the final visited words.
template <typename T>
__global__ void __launch_bounds__(BLOCK) msum_kernel(BatchArgs<T> a, unsigned long long *m_out) {
  constexpr int W = WordBits<T>::value;
  constexpr int PIECES = W / 32;
  __shared__ unsigned long long s_m[W];
  const int g = blockIdx.y;
  const int tid = threadIdx.x, lane = tid & 31;
  for (int j = tid; j < W; j += BLOCK) s_m[j] = 0;
  __syncthreads();
  const T *vis = a.visited + (size_t)g * a.gstride;
  const size_t stride = (size_t)gridDim.x * BLOCK;
  for (size_t base = (size_t)blockIdx.x * BLOCK; base < a.nv; base += stride) {
    const size_t v = base + tid;
    const bool in = v < a.nv;
    const T vv = in ? ld(vis + v) : wzero_value<T>();
    const uint32_t d = in ? __ldg(a.deg + v) : 0u;
#pragma unroll
    for (int k = 0; k < PIECES; ++k) {
      const uint32_t p = wpiece(vv, k);
      uint32_t any = __reduce_or_sync(FULL, p);
      while (any) {
        const int j = __ffs(any) - 1;
        any &= any - 1;
        const uint32_t x = ((p >> j) & 1u) ? d : 0u;
        const unsigned long long s =
            (unsigned long long)__reduce_add_sync(FULL, x & 0xffffu) +
            ((unsigned long long)__reduce_add_sync(FULL, x >> 16) << 16);
        if (lane == 0) atomicAdd(&s_m[k * 32 + j], s);
      }
    }
  }
  __syncthreads();
  const int rows = group_rows(a, g);
  for (int j = tid; j < rows; j += BLOCK)
    if (s_m[j]) atomicAdd(&m_out[(size_t)g * W + j], s_m[j]);
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
