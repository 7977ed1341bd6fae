// ibfs.cu -- C ABI of libibfs.so (include/ibfs.h): graph loading, the batch/level loop
// around the sm_100a kernels of kernels.cuh, statistics, allocator hook.
//
// Host orchestration of one ibfs_run_ex call:
//   groups = consecutive chunks of group_bits sources; G groups run per launch batch
//   (all of a batch's groups share each level launch; each keeps its own direction).
//   per batch: init_state + init_sources, then per level l = 1, 2, ...:
//     level_kernel(l) -- one cooperative launch: commit of level l-1, grid barrier,
//     expand of level l (kernels.cuh); every LEVELS_PER_CHECK levels the batch's
//     done-counter is copied to pinned host memory, with one chunk of look-ahead so the
//     device never waits for the host; kernels of a finished batch exit immediately.
//   then m_s (+ digest) finalize outside the timed window; D2H of rows if the caller's
//   buffer is on the host.
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_segmented_sort.cuh>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <exception>
#include <cstdio>
#include <cstring>
#include <cstdlib>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "../../include/ibfs.h"
#include "kernels.cuh"
#include "joint.cuh"
#include "plan.h"

using namespace ibfs;

// ------------------------------------------------------------------ error plumbing ----
namespace {
thread_local std::string g_last_error;

struct IbfsError {
  int code;
  std::string msg;
};

[[noreturn]] void fail(int code, const std::string &msg) { throw IbfsError{code, msg}; }

void cuda_check(cudaError_t e, const char *what) {
  if (e != cudaSuccess) {
    cudaGetLastError();
    int code = (e == cudaErrorMemoryAllocation) ? IBFS_E_NOMEM : IBFS_E_CUDA;
    fail(code, std::string(what) + ": " + cudaGetErrorString(e));
  }
}
#define CK(x) cuda_check((x), #x)

template <typename F>
int guarded(F &&f) {
  try {
    f();
    g_last_error.clear();
    return IBFS_OK;
  } catch (const IbfsError &e) {
    g_last_error = e.msg;
    return e.code;
  } catch (const std::bad_alloc &) {
    g_last_error = "host allocation failed";
    return IBFS_E_NOMEM;
  } catch (...) {
    g_last_error = "unknown internal error";
    return IBFS_E_CUDA;
  }
}

// Restores the caller's current device on scope exit.
struct DeviceScope {
  int prev = -1;
  explicit DeviceScope(int dev) {
    static const int n = [] {
      int c = 0;
      if (cudaGetDeviceCount(&c) != cudaSuccess) { cudaGetLastError(); c = 0; }
      return c;
    }();
    if (n == 0) fail(IBFS_E_CUDA, "no CUDA device available (libibfs has no CPU fallback)");
    if (dev < 0 || dev >= n) fail(IBFS_E_INVALID, "device index out of range");
    CK(cudaGetDevice(&prev));
    CK(cudaSetDevice(dev));
  }
  ~DeviceScope() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

// ------------------------------------------------------------------------ memory ----
struct Allocator {
  void *(*alloc)(size_t, int, void *) = nullptr;
  void (*release)(void *, int, void *) = nullptr;
  void *ctx = nullptr;
};
std::mutex g_alloc_mu;
Allocator g_alloc;

Allocator current_allocator() {
  std::lock_guard<std::mutex> lk(g_alloc_mu);
  return g_alloc;
}

// Scratch buffers kept by a graph between calls (the same call shape asks for the same
// buffers in the same order): a call that finds the cache free takes it for its whole
// duration and reuses buffer i for its i-th request when it is large enough; a concurrent
// call on the same graph finds it taken and allocates its own.  Saves the per-call
// allocate / free round trips (tens of them) between back-to-back calls.
struct ScratchCache {
  std::mutex mu;
  std::vector<std::pair<void *, size_t>> bufs;
  std::vector<char> zero;  // buffer i is known to be all zero (the clean ring)
  ~ScratchCache() {
    for (auto &b : bufs) cudaFree(b.first);
  }
};

// Device scratch owned by one call: caller allocator if installed, else the graph's cache
// when free, else the stream-ordered pool (cudaMallocAsync; the pool keeps memory across
// calls).
class Scratch {
 public:
  Scratch(int dev, cudaStream_t s, ScratchCache *cache = nullptr)
      : dev_(dev), stream_(s), al_(current_allocator()) {
    if (cache && !al_.alloc && cache->mu.try_lock()) cache_ = cache;
  }
  ~Scratch() {
    if (cache_) {
      // an exception left work in flight on the cached buffers: finish it before the next
      // call may reuse them
      if (std::uncaught_exceptions() > 0) cudaStreamSynchronize(stream_);
      cache_->mu.unlock();
      return;
    }
    for (void *p : ptrs_) {
      if (al_.alloc) al_.release(p, dev_, al_.ctx);
      else cudaFreeAsync(p, stream_);
    }
  }
  // A buffer that must be all zero: from the cache when the previous call left it zero
  // (mark_zero), else cleared here on the stream.  Returns its cache index (or -1).
  template <typename T>
  T *get_zeroed(size_t count, int *idx) {
    const size_t i = next_;
    const bool was_zero = cache_ && i < cache_->zero.size() && cache_->zero[i] && i < cache_->bufs.size() &&
                          cache_->bufs[i].second >= std::max<size_t>(count * sizeof(T), 256);
    T *p = get<T>(count);  // clears the flag
    // the whole allocation (a cached buffer may be larger than this request; a later call
    // may use more of it while the flag says zero)
    const size_t whole = cache_ ? cache_->bufs[i].second : std::max<size_t>(count * sizeof(T), 256);
    if (!was_zero) CK(cudaMemsetAsync(p, 0, whole, stream_));
    *idx = cache_ ? (int)i : -1;
    return p;
  }
  // the call leaves buffer idx all zero again (only after its work completed normally)
  void mark_zero(int idx) {
    if (!cache_ || idx < 0) return;
    if (cache_->zero.size() <= (size_t)idx) cache_->zero.resize(idx + 1, 0);
    cache_->zero[idx] = 1;
  }
  template <typename T>
  T *get(size_t count) {
    size_t bytes = std::max<size_t>(count * sizeof(T), 256);
    void *p = nullptr;
    if (cache_) {
      const size_t i = next_++;
      if (i < cache_->zero.size()) cache_->zero[i] = 0;  // handed out: contents unknown from now
      if (i < cache_->bufs.size() && cache_->bufs[i].second >= bytes) return static_cast<T *>(cache_->bufs[i].first);
      if (i < cache_->bufs.size()) {  // too small: replace (the previous call has completed)
        cudaFree(cache_->bufs[i].first);
        cache_->bufs[i] = {nullptr, 0};
      }
      bytes = (bytes + (1u << 20) - 1) & ~(size_t)((1u << 20) - 1);  // round up: fewer regrowths
      cudaError_t e = cudaMalloc(&p, bytes);
      if (e != cudaSuccess) {
        cudaGetLastError();
        fail(IBFS_E_NOMEM, "cudaMalloc(" + std::to_string(bytes) + " bytes) failed");
      }
      if (i < cache_->bufs.size()) cache_->bufs[i] = {p, bytes};
      else cache_->bufs.push_back({p, bytes});
      return static_cast<T *>(p);
    }
    if (al_.alloc) {
      p = al_.alloc(bytes, dev_, al_.ctx);
      if (!p) fail(IBFS_E_NOMEM, "caller allocator returned NULL");
    } else {
      cudaError_t e = cudaMallocAsync(&p, bytes, stream_);
      if (e != cudaSuccess) {
        cudaGetLastError();
        fail(IBFS_E_NOMEM, "cudaMallocAsync(" + std::to_string(bytes) + " bytes) failed");
      }
    }
    ptrs_.push_back(p);
    return static_cast<T *>(p);
  }

 private:
  int dev_;
  cudaStream_t stream_;
  Allocator al_;
  std::vector<void *> ptrs_;
  ScratchCache *cache_ = nullptr;
  size_t next_ = 0;
};

void set_pool_threshold(int dev) {
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  cudaGetLastError();
}

bool is_device_ptr(const void *p) {
  if (!p) return false;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
}

}  // namespace

// -------------------------------------------------------------------------- graph ----
// The device graph lives in a compacted vertex space: the vertices of degree > 0, in the
// caller's id order (compacted id = rank among them).  Isolated vertices never hold a
// status word, never enter a queue and are never read by a level kernel; their depth
// rows are written directly (-1, or 0 at an isolated source).  Because the ranks keep
// the caller's order, adjacency rows keep their order and every "lower id" tie-break is
// unchanged.
struct ibfs_graph {
  int device = 0;
  uint32_t nv = 0;          // caller's vertices
  uint32_t nva = 0;         // vertices of degree > 0 (the compacted space)
  uint64_t ne = 0;
  uint32_t max_deg = 0;
  uint64_t nv_active = 0;   // = nva
  unsigned long long *d_off = nullptr;  // [nva + 1]
  uint32_t *d_adj = nullptr;            // [ne] compacted ids
  uint32_t *d_deg = nullptr;            // [nva]
  uint32_t *d_tbase = nullptr;          // [nv/128 + 1]: vertices of degree > 0 before tile t
  uint32_t *d_nzbits = nullptr;         // [nv/32]: bit v%32 of word v/32 = (deg(v) > 0)
  HubChunk *d_chunks = nullptr;
  uint32_t n_chunks = 0;
  uint32_t *d_hub_vtx = nullptr;     // [n_hubs] vertices of degree > HUB_T (ascending)
  uint32_t *d_hub_chunk0 = nullptr;  // [n_hubs + 1] first chunk of each hub
  uint32_t n_hubs = 0;
  std::vector<uint64_t> h_off;      // host copy of d_off (tiling, planner)
  // Directed graphs ("store the reverse edges" for bottom-up): the in-edge CSR in
  // the same compacted space (a vertex is kept if it has an out- or an in-edge), with its
  // own degrees and hub chunks.  Undirected: directed = false and none of these is
  // allocated (the kernels read the out-edge arrays for both directions).
  bool directed = false;
  unsigned long long *d_roff = nullptr;
  uint32_t *d_radj = nullptr;
  uint32_t *d_rdeg = nullptr;
  HubChunk *d_rchunks = nullptr;
  uint32_t n_rchunks = 0;
  uint32_t *d_rhub_vtx = nullptr;
  uint32_t *d_rhub_chunk0 = nullptr;
  uint32_t n_rhubs = 0;
  std::vector<uint64_t> h_roff;
  std::vector<uint32_t> h_tbase, h_nzbits;
  int num_sms = 148;
  size_t total_mem = 0;  // device memory (bytes), queried once at load
  int level_blocks_per_sm[3] = {1, 1, 1};  // co-resident level_kernel CTAs per SM (W = 32, 64, 128)
  int dtma_blocks_per_sm[3] = {1, 1, 1};   // depth_tma_kernel (grid = SMs x this / groups)
  int depth_blocks_per_sm[3] = {1, 1, 1};  // depth_kernel
  ScratchCache scratch;  // run scratch kept between calls (Scratch)
};

namespace {

void graph_release(ibfs_graph *g) {
  if (!g) return;
  int prev = -1;
  if (cudaGetDevice(&prev) == cudaSuccess) cudaSetDevice(g->device);
  cudaFree(g->d_off);
  cudaFree(g->d_adj);
  cudaFree(g->d_deg);
  cudaFree(g->d_chunks);
  cudaFree(g->d_hub_vtx);
  cudaFree(g->d_hub_chunk0);
  cudaFree(g->d_tbase);
  cudaFree(g->d_nzbits);
  cudaFree(g->d_roff);
  cudaFree(g->d_radj);
  cudaFree(g->d_rdeg);
  cudaFree(g->d_rchunks);
  cudaFree(g->d_rhub_vtx);
  cudaFree(g->d_rhub_chunk0);
  {
    std::lock_guard<std::mutex> lk(g->scratch.mu);
    for (auto &b : g->scratch.bufs) cudaFree(b.first);
    g->scratch.bufs.clear();
  }
  if (prev >= 0) cudaSetDevice(prev);
  cudaGetLastError();
  delete g;
}

__global__ void degree_kernel(const unsigned long long *off, uint32_t nv, uint32_t *deg,
                              unsigned long long *maxdeg_nz) {
  uint32_t local_max = 0, local_nz = 0;
  for (size_t v = (size_t)blockIdx.x * blockDim.x + threadIdx.x; v < nv;
       v += (size_t)gridDim.x * blockDim.x) {
    unsigned long long d = off[v + 1] - off[v];
    uint32_t d32 = d > 0xffffffffull ? 0xffffffffu : (uint32_t)d;
    deg[v] = d32;
    local_max = max(local_max, d32);
    local_nz += d32 > 0;
  }
  local_max = __reduce_max_sync(FULL, local_max);
  local_nz = __reduce_add_sync(FULL, local_nz);
  if ((threadIdx.x & 31) == 0) {
    atomicMax(&maxdeg_nz[0], (unsigned long long)local_max);
    atomicAdd(&maxdeg_nz[1], (unsigned long long)local_nz);
  }
}

__global__ void max_id_kernel(const uint32_t *adj, unsigned long long ne, uint32_t *mx) {
  uint32_t m = 0;
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < ne;
       i += (unsigned long long)gridDim.x * blockDim.x)
    m = max(m, adj[i]);
  m = __reduce_max_sync(FULL, m);
  if ((threadIdx.x & 31) == 0) atomicMax(mx, m);
}

// ---- compaction ----
// a vertex is kept when it has an out-edge or (directed, roff != NULL) an in-edge
__global__ void nzbits_kernel(const unsigned long long *off, const unsigned long long *roff, uint32_t nv,
                              uint32_t *nzbits) {
  const size_t nvr = ((size_t)nv + 31) & ~(size_t)31;
  for (size_t v = (size_t)blockIdx.x * blockDim.x + threadIdx.x; v < nvr; v += (size_t)gridDim.x * blockDim.x) {
    const bool nz = v < nv && (off[v + 1] > off[v] || (roff && roff[v + 1] > roff[v]));
    const uint32_t b = __ballot_sync(FULL, nz);
    if ((threadIdx.x & 31) == 0) nzbits[v >> 5] = b;
  }
}

__global__ void tilecount_kernel(const uint32_t *nzbits, uint32_t nwords, uint32_t ntiles, uint32_t *cnt) {
  for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t < ntiles; t += gridDim.x * blockDim.x) {
    uint32_t c = 0;
    for (uint32_t k = 4 * t; k < min(4 * t + 4, nwords); ++k) c += __popc(nzbits[k]);
    cnt[t] = c;
  }
}

__device__ __forceinline__ uint32_t dev_compact_id(const uint32_t *tbase, const uint32_t *nzbits, uint32_t v) {
  const uint32_t w = v >> 5;
  uint32_t c = tbase[v >> 7];
  for (uint32_t k = w & ~3u; k < w; ++k) c += __popc(nzbits[k]);
  return c + __popc(nzbits[w] & ((1u << (v & 31)) - 1u));
}

// the run's sources in compacted ids (NO_VERTEX for an isolated source)
__global__ void compact_sources_kernel(const uint32_t *src, uint32_t n, const uint32_t *tbase, const uint32_t *nzbits,
                                       uint32_t *csrc) {
  for (uint32_t r = blockIdx.x * blockDim.x + threadIdx.x; r < n; r += gridDim.x * blockDim.x) {
    const uint32_t v = src[r];
    csrc[r] = ((nzbits[v >> 5] >> (v & 31)) & 1u) ? dev_compact_id(tbase, nzbits, v) : NO_VERTEX;
  }
}

__global__ void compact_rows_kernel(const unsigned long long *off, uint32_t nv, const uint32_t *tbase,
                                    const uint32_t *nzbits, unsigned long long *off_c) {
  for (size_t v = (size_t)blockIdx.x * blockDim.x + threadIdx.x; v < nv; v += (size_t)gridDim.x * blockDim.x) {
    if ((nzbits[v >> 5] >> (v & 31)) & 1u) off_c[dev_compact_id(tbase, nzbits, (uint32_t)v)] = off[v];
  }
}

__global__ void remap_adj_kernel(uint32_t *adj, unsigned long long ne, const uint32_t *tbase, const uint32_t *nzbits) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < ne;
       i += (unsigned long long)gridDim.x * blockDim.x)
    adj[i] = dev_compact_id(tbase, nzbits, adj[i]);
}

// d_off_orig [nv + 1] (caller ids, consumed and freed) and g->d_adj (caller ids, remapped in
// place) -> compacted g->d_off, g->d_adj, g->d_tbase, g->d_nzbits, host copies; for a
// directed graph the same for d_roff_orig / g->d_radj -> g->d_roff, g->d_radj.
void compact_graph(ibfs_graph *g, unsigned long long *d_off_orig, unsigned long long *d_roff_orig = nullptr) {
  const uint32_t nv = g->nv;
  const uint32_t nwords = (nv + 31) / 32, ntiles = (nv + 127) / 128;
  // padded to whole 128-vertex tiles (+1) so a tile's 4 words load as one uint4
  const size_t nz_alloc = ((size_t)ntiles + 1) * 4;
  CK(cudaMalloc(&g->d_nzbits, nz_alloc * 4));
  CK(cudaMemset(g->d_nzbits, 0, nz_alloc * 4));
  CK(cudaMalloc(&g->d_tbase, ((size_t)ntiles + 1) * 4));
  uint32_t *cnt = nullptr;
  void *tmp = nullptr;
  try {
    CK(cudaMalloc(&cnt, ((size_t)ntiles + 1) * 4));
    CK(cudaMemset(cnt, 0, ((size_t)ntiles + 1) * 4));
    nzbits_kernel<<<2048, 256>>>(d_off_orig, d_roff_orig, nv, g->d_nzbits);
    tilecount_kernel<<<(ntiles + 255) / 256, 256>>>(g->d_nzbits, nwords, ntiles, cnt);
    CK(cudaGetLastError());
    size_t tb = 0;
    CK(cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, g->d_tbase, (int64_t)ntiles + 1));
    CK(cudaMalloc(&tmp, std::max<size_t>(tb, 256)));
    CK(cub::DeviceScan::ExclusiveSum(tmp, tb, cnt, g->d_tbase, (int64_t)ntiles + 1));
    g->h_tbase.resize((size_t)ntiles + 1);
    g->h_nzbits.resize(nwords);
    CK(cudaMemcpy(g->h_tbase.data(), g->d_tbase, ((size_t)ntiles + 1) * 4, cudaMemcpyDeviceToHost));
    if (nwords) CK(cudaMemcpy(g->h_nzbits.data(), g->d_nzbits, (size_t)nwords * 4, cudaMemcpyDeviceToHost));
    g->nva = g->h_tbase[ntiles];
    CK(cudaMalloc(&g->d_off, ((size_t)g->nva + 1) * sizeof(unsigned long long)));
    const unsigned long long ne = g->ne;
    CK(cudaMemcpy(g->d_off + g->nva, &ne, sizeof(ne), cudaMemcpyHostToDevice));
    compact_rows_kernel<<<2048, 256>>>(d_off_orig, nv, g->d_tbase, g->d_nzbits, g->d_off);
    if (g->ne) remap_adj_kernel<<<4096, 256>>>(g->d_adj, g->ne, g->d_tbase, g->d_nzbits);
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
  } catch (...) {
    cudaFree(cnt);
    cudaFree(tmp);
    cudaFree(d_off_orig);
    cudaFree(d_roff_orig);
    throw;
  }
  cudaFree(cnt);
  cudaFree(tmp);
  cudaFree(d_off_orig);
  g->h_off.resize((size_t)g->nva + 1);
  CK(cudaMemcpy(g->h_off.data(), g->d_off, ((size_t)g->nva + 1) * 8, cudaMemcpyDeviceToHost));
  if (d_roff_orig) {
    try {
      CK(cudaMalloc(&g->d_roff, ((size_t)g->nva + 1) * sizeof(unsigned long long)));
      const unsigned long long ne = g->ne;
      CK(cudaMemcpy(g->d_roff + g->nva, &ne, sizeof(ne), cudaMemcpyHostToDevice));
      compact_rows_kernel<<<2048, 256>>>(d_roff_orig, g->nv, g->d_tbase, g->d_nzbits, g->d_roff);
      if (g->ne) remap_adj_kernel<<<4096, 256>>>(g->d_radj, g->ne, g->d_tbase, g->d_nzbits);
      CK(cudaGetLastError());
      CK(cudaDeviceSynchronize());
    } catch (...) {
      cudaFree(d_roff_orig);
      throw;
    }
    cudaFree(d_roff_orig);
    g->h_roff.resize((size_t)g->nva + 1);
    CK(cudaMemcpy(g->h_roff.data(), g->d_roff, ((size_t)g->nva + 1) * 8, cudaMemcpyDeviceToHost));
  }
}

// Host twin of compact_id for a caller id; NO_VERTEX if the vertex is isolated.
uint32_t host_compact_id(const ibfs_graph *g, uint32_t v) {
  const uint32_t w = v >> 5;
  const uint32_t bits = g->h_nzbits[w];
  if (!((bits >> (v & 31)) & 1u)) return NO_VERTEX;
  uint32_t c = g->h_tbase[v >> 7];
  for (uint32_t k = w & ~3u; k < w; ++k) c += (uint32_t)__builtin_popcount(g->h_nzbits[k]);
  return c + (uint32_t)__builtin_popcount(bits & ((1u << (v & 31)) - 1u));
}

// Static hub decomposition: the rows of vertices with degree > HUB_T are
// cut into chunks of CHUNK edges, each a work item a whole CTA sweeps.
void build_decomposition(const std::vector<uint64_t> &h_off, uint32_t nva, HubChunk **d_chunks,
                         uint32_t *n_chunks, uint32_t **d_hub_vtx, uint32_t **d_hub_chunk0, uint32_t *n_hubs) {
  std::vector<HubChunk> chunks;
  std::vector<uint32_t> hubs, chunk0;
  for (uint32_t v = 0; v < nva; ++v) {
    const uint64_t d = h_off[v + 1] - h_off[v];
    if (d <= (uint64_t)HUB_T) continue;
    hubs.push_back(v);
    chunk0.push_back((uint32_t)chunks.size());
    uint32_t first = 1;
    for (uint64_t e = h_off[v]; e < h_off[v + 1]; e += CHUNK) {
      HubChunk c;
      c.e0 = e;
      c.e1 = std::min<uint64_t>(e + CHUNK, h_off[v + 1]);
      c.v = v;
      c.first = first;
      first = 0;
      chunks.push_back(c);
    }
  }
  *n_chunks = (uint32_t)chunks.size();
  chunk0.push_back(*n_chunks);
  *n_hubs = (uint32_t)hubs.size();
  CK(cudaMalloc(d_chunks, std::max<size_t>(chunks.size(), 1) * sizeof(HubChunk)));
  if (!chunks.empty())
    CK(cudaMemcpy(*d_chunks, chunks.data(), chunks.size() * sizeof(HubChunk), cudaMemcpyHostToDevice));
  CK(cudaMalloc(d_hub_vtx, std::max<size_t>(hubs.size(), 1) * 4));
  CK(cudaMalloc(d_hub_chunk0, chunk0.size() * 4));
  if (!hubs.empty()) CK(cudaMemcpy(*d_hub_vtx, hubs.data(), hubs.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(*d_hub_chunk0, chunk0.data(), chunk0.size() * 4, cudaMemcpyHostToDevice));
}

// Degrees, max degree, hub chunks; compacted offsets must be in g->d_off and g->h_off.
void finish_graph(ibfs_graph *g) {
  CK(cudaMalloc(&g->d_deg, std::max<size_t>(g->nva, 1) * sizeof(uint32_t)));
  unsigned long long *d_stats = nullptr;
  CK(cudaMalloc(&d_stats, 2 * sizeof(unsigned long long)));
  CK(cudaMemset(d_stats, 0, 2 * sizeof(unsigned long long)));
  degree_kernel<<<1024, 256>>>(g->d_off, g->nva, g->d_deg, d_stats);
  CK(cudaGetLastError());
  unsigned long long h[2];
  CK(cudaMemcpy(h, d_stats, sizeof(h), cudaMemcpyDeviceToHost));
  cudaFree(d_stats);
  for (uint32_t v = 0; v < g->nva; ++v)
    if (g->h_off[v + 1] - g->h_off[v] > 0xffffffffull)
      fail(IBFS_E_UNSUPPORTED, "vertex degree >= 2^32");
  g->max_deg = (uint32_t)h[0];
  g->nv_active = h[1];
  build_decomposition(g->h_off, g->nva, &g->d_chunks, &g->n_chunks, &g->d_hub_vtx, &g->d_hub_chunk0, &g->n_hubs);
  if (g->directed) {
    CK(cudaMalloc(&g->d_rdeg, std::max<size_t>(g->nva, 1) * sizeof(uint32_t)));
    CK(cudaMalloc(&d_stats, 2 * sizeof(unsigned long long)));
    CK(cudaMemset(d_stats, 0, 2 * sizeof(unsigned long long)));
    degree_kernel<<<1024, 256>>>(g->d_roff, g->nva, g->d_rdeg, d_stats);
    CK(cudaGetLastError());
    CK(cudaMemcpy(h, d_stats, sizeof(h), cudaMemcpyDeviceToHost));
    cudaFree(d_stats);
    for (uint32_t v = 0; v < g->nva; ++v)
      if (g->h_roff[v + 1] - g->h_roff[v] > 0xffffffffull) fail(IBFS_E_UNSUPPORTED, "vertex in-degree >= 2^32");
    build_decomposition(g->h_roff, g->nva, &g->d_rchunks, &g->n_rchunks, &g->d_rhub_vtx, &g->d_rhub_chunk0,
                        &g->n_rhubs);
  }
  int dev = g->device;
  CK(cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, dev));
  {
    size_t free_b = 0;
    CK(cudaMemGetInfo(&free_b, &g->total_mem));
  }
  CK(cudaFuncSetAttribute(level_kernel<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)sizeof(TileQueue<uint32_t>)));
  CK(cudaFuncSetAttribute(level_kernel<unsigned long long>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)sizeof(TileQueue<unsigned long long>)));
  CK(cudaFuncSetAttribute(level_kernel<u128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)sizeof(TileQueue<u128>)));
  CK(cudaFuncSetAttribute(depth_kernel<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)depth_smem_bytes<uint32_t>()));
  CK(cudaFuncSetAttribute(depth_kernel<unsigned long long>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)depth_smem_bytes<unsigned long long>()));
  CK(cudaFuncSetAttribute(depth_kernel<u128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)depth_smem_bytes<u128>()));
  CK(cudaFuncSetAttribute(depth_tma_kernel<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)depth_tma_smem_bytes<uint32_t>()));
  CK(cudaFuncSetAttribute(depth_tma_kernel<unsigned long long>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)depth_tma_smem_bytes<unsigned long long>()));
  CK(cudaFuncSetAttribute(depth_tma_kernel<u128>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                          (int)depth_tma_smem_bytes<u128>()));
  int occ = 1;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, level_kernel<uint32_t>, BLOCK, sizeof(TileQueue<uint32_t>)));
  g->level_blocks_per_sm[0] = std::max(1, occ);
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, level_kernel<unsigned long long>, BLOCK,
                                                   sizeof(TileQueue<unsigned long long>)));
  g->level_blocks_per_sm[1] = std::max(1, occ);
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, level_kernel<u128>, BLOCK, sizeof(TileQueue<u128>)));
  g->level_blocks_per_sm[2] = std::max(1, occ);
  // the depth kernels are persistent over their tiles: their grids are sized from the
  // occupancy the shared-memory footprint really allows (not from the launch bounds)
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, depth_tma_kernel<uint32_t>, DTHREADS + 32,
                                                   depth_tma_smem_bytes<uint32_t>()));
  g->dtma_blocks_per_sm[0] = std::max(1, occ);
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, depth_tma_kernel<unsigned long long>, DTHREADS + 32,
                                                   depth_tma_smem_bytes<unsigned long long>()));
  g->dtma_blocks_per_sm[1] = std::max(1, occ);
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, depth_tma_kernel<u128>, DTHREADS + 32,
                                                   depth_tma_smem_bytes<u128>()));
  g->dtma_blocks_per_sm[2] = std::max(1, occ);
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, depth_kernel<uint32_t>, DTHREADS + 32,
                                                   depth_smem_bytes<uint32_t>()));
  g->depth_blocks_per_sm[0] = std::max(1, occ);
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, depth_kernel<unsigned long long>, DTHREADS + 32,
                                                   depth_smem_bytes<unsigned long long>()));
  g->depth_blocks_per_sm[1] = std::max(1, occ);
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, depth_kernel<u128>, DTHREADS + 32, depth_smem_bytes<u128>()));
  g->depth_blocks_per_sm[2] = std::max(1, occ);
  if (std::getenv("IBFS_VERBOSE"))
    std::fprintf(stderr, "ibfs: CTAs/SM level %d/%d/%d depth_tma %d/%d/%d depth %d/%d/%d (W=32/64/128); smem depth_tma %zu B\n",
                 g->level_blocks_per_sm[0], g->level_blocks_per_sm[1], g->level_blocks_per_sm[2],
                 g->dtma_blocks_per_sm[0], g->dtma_blocks_per_sm[1], g->dtma_blocks_per_sm[2],
                 g->depth_blocks_per_sm[0], g->depth_blocks_per_sm[1], g->depth_blocks_per_sm[2],
                 depth_tma_smem_bytes<u128>());
  set_pool_threshold(dev);
}

// undirected tuple (a, b) -> CSR entries a->b and b->a
__global__ void explode_kernel(const uint32_t *u, const uint32_t *v, unsigned long long m, uint32_t *keys,
                               uint32_t *vals) {
  for (unsigned long long e = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; e < m;
       e += (unsigned long long)gridDim.x * blockDim.x) {
    const uint32_t a = u[e], b = v[e];
    keys[2 * e] = a;
    vals[2 * e] = b;
    keys[2 * e + 1] = b;
    vals[2 * e + 1] = a;
  }
}

__global__ void check_ids_kernel(const uint32_t *u, const uint32_t *v, unsigned long long m, uint32_t nv,
                                 uint32_t *bad) {
  for (unsigned long long e = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; e < m;
       e += (unsigned long long)gridDim.x * blockDim.x)
    if (u[e] >= nv || v[e] >= nv) *bad = 1;
}

__global__ void count_ids_kernel(const uint32_t *adj, unsigned long long ne, unsigned long long *cnt) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < ne;
       i += (unsigned long long)gridDim.x * blockDim.x)
    atomicAdd(cnt + adj[i], 1ull);
}

// occurrences of every id in adj[ne] == the row lengths of the other CSR side (h_off)
bool degrees_match(const uint32_t *d_adj, uint64_t ne, const std::vector<uint64_t> &h_off, uint32_t nv) {
  unsigned long long *cnt = nullptr;
  CK(cudaMalloc(&cnt, (size_t)nv * 8));
  std::vector<unsigned long long> h(nv);
  try {
    CK(cudaMemset(cnt, 0, (size_t)nv * 8));
    count_ids_kernel<<<4096, 256>>>(d_adj, ne, cnt);
    CK(cudaGetLastError());
    CK(cudaMemcpy(h.data(), cnt, (size_t)nv * 8, cudaMemcpyDeviceToHost));
  } catch (...) {
    cudaFree(cnt);
    throw;
  }
  cudaFree(cnt);
  for (uint32_t v = 0; v < nv; ++v)
    if (h[v] != h_off[v + 1] - h_off[v]) return false;
  return true;
}

}  // namespace

extern "C" int ibfs_version(void) { return 10000; }

extern "C" const char *ibfs_last_error(void) { return g_last_error.c_str(); }

extern "C" int ibfs_load_csr(int device, uint32_t nv, uint64_t ne, const uint64_t *offsets,
                             const uint32_t *adj, const uint64_t *rev_offsets,
                             const uint32_t *rev_adj, ibfs_graph **out_graph) {
  return guarded([&] {
    if (!out_graph) fail(IBFS_E_INVALID, "out_graph is NULL");
    *out_graph = nullptr;
    if (nv == 0) fail(IBFS_E_INVALID, "nv must be >= 1");
    if (!offsets || (ne > 0 && !adj)) fail(IBFS_E_INVALID, "offsets/adj is NULL");
    if (ne >= (1ull << 40)) fail(IBFS_E_INVALID, "ne too large");
    const bool directed = rev_offsets != nullptr;
    if (directed != (rev_adj != nullptr) && ne > 0) fail(IBFS_E_INVALID, "rev_offsets and rev_adj must both be set");
    DeviceScope ds(device);
    ibfs_graph *g = new ibfs_graph();
    unsigned long long *d_off_orig = nullptr, *d_roff_orig = nullptr;
    // one CSR side: validate the offsets on the host, copy both arrays, check the ids
    auto load_side = [&](const uint64_t *o, const uint32_t *ad, std::vector<uint64_t> &h, unsigned long long **d_o,
                         uint32_t **d_a) {
      h.resize((size_t)nv + 1);
      CK(cudaMemcpy(h.data(), o, ((size_t)nv + 1) * sizeof(uint64_t), cudaMemcpyDefault));
      if (h[0] != 0 || h[nv] != ne) fail(IBFS_E_INVALID, "offsets[0] != 0 or offsets[nv] != ne");
      for (uint32_t v = 0; v < nv; ++v)
        if (h[v + 1] < h[v]) fail(IBFS_E_INVALID, "offsets not non-decreasing");
      CK(cudaMalloc(d_o, ((size_t)nv + 1) * sizeof(unsigned long long)));
      CK(cudaMemcpy(*d_o, h.data(), ((size_t)nv + 1) * sizeof(uint64_t), cudaMemcpyHostToDevice));
      CK(cudaMalloc(d_a, std::max<uint64_t>(ne, 1) * sizeof(uint32_t)));
      if (ne) {
        CK(cudaMemcpy(*d_a, ad, ne * sizeof(uint32_t), cudaMemcpyDefault));
        uint32_t *d_mx = nullptr;
        CK(cudaMalloc(&d_mx, sizeof(uint32_t)));
        CK(cudaMemset(d_mx, 0, sizeof(uint32_t)));
        max_id_kernel<<<1024, 256>>>(*d_a, ne, d_mx);
        CK(cudaGetLastError());
        uint32_t mx = 0;
        CK(cudaMemcpy(&mx, d_mx, sizeof(uint32_t), cudaMemcpyDeviceToHost));
        cudaFree(d_mx);
        if (mx >= nv) fail(IBFS_E_INVALID, "adjacency id >= nv");
      }
    };
    try {
      g->device = device;
      g->nv = nv;
      g->ne = ne;
      g->directed = directed;
      load_side(offsets, adj, g->h_off, &d_off_orig, &g->d_adj);
      if (directed) {
        load_side(rev_offsets, rev_adj, g->h_roff, &d_roff_orig, &g->d_radj);
        // the in-edge CSR must be the transpose: every vertex's in-degree (its
        // occurrences in adj) equals its reverse row length, and vice versa
        if (ne && (!degrees_match(g->d_adj, ne, g->h_roff, nv) || !degrees_match(g->d_radj, ne, g->h_off, nv)))
          fail(IBFS_E_INVALID, "rev_offsets/rev_adj is not the transpose of offsets/adj");
      }
      unsigned long long *o = d_off_orig, *ro = d_roff_orig;
      d_off_orig = d_roff_orig = nullptr;
      compact_graph(g, o, ro);  // frees o and ro
      finish_graph(g);
    } catch (...) {
      cudaFree(d_off_orig);
      cudaFree(d_roff_orig);
      graph_release(g);
      throw;
    }
    *out_graph = g;
  });
}

extern "C" int ibfs_load_edges(int device, uint32_t nv, uint64_t n_tuples, const uint32_t *u,
                               const uint32_t *v, int directed, ibfs_graph **out_graph) {
  return guarded([&] {
    if (!out_graph) fail(IBFS_E_INVALID, "out_graph is NULL");
    *out_graph = nullptr;
    if (nv == 0) fail(IBFS_E_INVALID, "nv must be >= 1");
    if (n_tuples > 0 && (!u || !v)) fail(IBFS_E_INVALID, "u/v is NULL");
    if (n_tuples >= (1ull << 39)) fail(IBFS_E_INVALID, "too many tuples");
    DeviceScope ds(device);
    // undirected: tuple (u, v) -> entries u->v and v->u; directed: u->v only, plus
    // the in-edge rows v <- u for bottom-up
    const uint64_t ne = directed ? n_tuples : 2 * n_tuples;
    ibfs_graph *g = new ibfs_graph();
    std::vector<void *> tmp;
    auto dalloc = [&](size_t bytes) {
      void *p = nullptr;
      CK(cudaMalloc(&p, std::max<size_t>(bytes, 256)));
      tmp.push_back(p);
      return p;
    };
    auto dfree = [&](void *p) {
      for (void *&q : tmp)
        if (q == p) q = nullptr;
      cudaFree(p);
    };
    int bits = 1;
    while (bits < 32 && (1ull << bits) < nv) ++bits;
    // rows of (key -> val) pairs: offsets = exclusive scan of the key histogram; a stable
    // radix sort by key keeps tuple order within each row
    auto build_rows = [&](const uint32_t *keys, const uint32_t *vals, uint64_t m, unsigned long long *off_out,
                          uint32_t *adj_out) {
      unsigned long long *deg = (unsigned long long *)dalloc(((size_t)nv + 1) * 8);
      CK(cudaMemset(deg, 0, ((size_t)nv + 1) * 8));
      if (m) {
        count_ids_kernel<<<4096, 256>>>(keys, m, deg);
        CK(cudaGetLastError());
      }
      size_t tb = 0;
      CK(cub::DeviceScan::ExclusiveSum(nullptr, tb, deg, off_out, (int64_t)nv + 1));
      void *t = dalloc(tb);
      CK(cub::DeviceScan::ExclusiveSum(t, tb, deg, off_out, (int64_t)nv + 1));
      if (m) {
        uint32_t *keys_out = (uint32_t *)dalloc(m * 4);
        size_t tb2 = 0;
        CK(cub::DeviceRadixSort::SortPairs(nullptr, tb2, keys, keys_out, vals, adj_out, (int64_t)m, 0, bits));
        void *t2 = dalloc(tb2);
        CK(cub::DeviceRadixSort::SortPairs(t2, tb2, keys, keys_out, vals, adj_out, (int64_t)m, 0, bits));
        CK(cudaDeviceSynchronize());
        dfree(keys_out);
        dfree(t2);
      }
      CK(cudaDeviceSynchronize());
      dfree(deg);
      dfree(t);
    };
    try {
      g->device = device;
      g->nv = nv;
      g->ne = ne;
      g->directed = directed != 0;
      uint32_t *d_u = (uint32_t *)dalloc(n_tuples * 4), *d_v = (uint32_t *)dalloc(n_tuples * 4);
      if (n_tuples) {
        CK(cudaMemcpy(d_u, u, n_tuples * 4, cudaMemcpyDefault));
        CK(cudaMemcpy(d_v, v, n_tuples * 4, cudaMemcpyDefault));
      }
      uint32_t *bad = (uint32_t *)dalloc(4);
      CK(cudaMemset(bad, 0, 4));
      if (n_tuples) {
        check_ids_kernel<<<4096, 256>>>(d_u, d_v, n_tuples, nv, bad);
        CK(cudaGetLastError());
      }
      uint32_t hbad = 0;
      CK(cudaMemcpy(&hbad, bad, 4, cudaMemcpyDeviceToHost));
      if (hbad) fail(IBFS_E_INVALID, "tuple vertex id >= nv");
      unsigned long long *d_off_orig = (unsigned long long *)dalloc(((size_t)nv + 1) * sizeof(unsigned long long));
      unsigned long long *d_roff_orig = nullptr;
      CK(cudaMalloc(&g->d_adj, std::max<uint64_t>(ne, 1) * sizeof(uint32_t)));
      if (directed) {
        d_roff_orig = (unsigned long long *)dalloc(((size_t)nv + 1) * sizeof(unsigned long long));
        CK(cudaMalloc(&g->d_radj, std::max<uint64_t>(ne, 1) * sizeof(uint32_t)));
        build_rows(d_u, d_v, n_tuples, d_off_orig, g->d_adj);   // out-edges u -> v
        build_rows(d_v, d_u, n_tuples, d_roff_orig, g->d_radj); // in-edges v <- u
      } else {
        uint32_t *keys_a = (uint32_t *)dalloc(ne * 4), *vals_a = (uint32_t *)dalloc(ne * 4);
        if (n_tuples) {
          explode_kernel<<<4096, 256>>>(d_u, d_v, n_tuples, keys_a, vals_a);
          CK(cudaGetLastError());
        }
        dfree(d_u);
        dfree(d_v);
        build_rows(keys_a, vals_a, ne, d_off_orig, g->d_adj);
      }
      CK(cudaDeviceSynchronize());
      for (void *&p : tmp)
        if (p && p != d_off_orig && p != d_roff_orig) { cudaFree(p); p = nullptr; }
      tmp.clear();
      compact_graph(g, d_off_orig, d_roff_orig);  // frees both
      finish_graph(g);
    } catch (...) {
      for (void *p : tmp) cudaFree(p);
      graph_release(g);
      throw;
    }
    *out_graph = g;
  });
}

namespace {
// key = ~deg(w): ascending key order = neighbour degree descending
__global__ void hubkey_kernel(const uint32_t *adj, const uint32_t *deg, unsigned long long n, uint32_t *keys) {
  for (unsigned long long i = (unsigned long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (unsigned long long)gridDim.x * blockDim.x)
    keys[i] = ~deg[adj[i]];
}
__global__ void rel_offsets_kernel(const unsigned long long *off, uint32_t r0, uint32_t nr, int *rel) {
  const unsigned long long base = off[r0];
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i <= nr; i += gridDim.x * blockDim.x)
    rel[i] = (int)(off[r0 + i] - base);
}
}  // namespace

extern "C" int ibfs_graph_sort_rows(ibfs_graph *g, int order) {
  return guarded([&] {
    if (!g) fail(IBFS_E_INVALID, "graph is NULL");
    if (order != IBFS_ROWS_KEEP && order != IBFS_ROWS_HUB_FIRST) fail(IBFS_E_INVALID, "bad row order");
    if (order == IBFS_ROWS_KEEP || g->ne == 0) return;
    DeviceScope ds(g->device);
    // the rows bottom-up scans: the in-edge rows of a directed graph, keyed
    // by the in-degree of the parent (a vertex with many in-edges is reached early)
    const std::vector<uint64_t> &h_off = g->directed ? g->h_roff : g->h_off;
    const unsigned long long *d_off = g->directed ? g->d_roff : g->d_off;
    uint32_t *d_adj = g->directed ? g->d_radj : g->d_adj;
    const uint32_t *d_kdeg = g->directed ? g->d_rdeg : g->d_deg;
    // rows in batches of <= 2^30 entries (CUB segmented sort takes int sizes)
    const unsigned long long cap = 1ull << 30;
    unsigned long long maxb = 0;
    std::vector<std::pair<uint32_t, uint32_t>> batches;
    uint32_t r0 = 0;
    while (r0 < g->nva) {
      uint32_t r1 = r0;
      while (r1 < g->nva && h_off[r1 + 1] - h_off[r0] <= cap) ++r1;
      if (r1 == r0) ++r1;  // a single row longer than cap (degree > 2^30): not expected
      batches.push_back({r0, r1});
      maxb = std::max<unsigned long long>(maxb, h_off[r1] - h_off[r0]);
      r0 = r1;
    }
    if (maxb > 0x7fffffffull) fail(IBFS_E_UNSUPPORTED, "row longer than 2^31 entries");
    std::vector<void *> tmp;
    auto dalloc = [&](size_t bytes) {
      void *p = nullptr;
      CK(cudaMalloc(&p, std::max<size_t>(bytes, 256)));
      tmp.push_back(p);
      return p;
    };
    try {
      uint32_t *kin = (uint32_t *)dalloc(maxb * 4), *kout = (uint32_t *)dalloc(maxb * 4);
      uint32_t *vout = (uint32_t *)dalloc(maxb * 4);
      size_t max_rows = 0;
      for (auto &b : batches) max_rows = std::max<size_t>(max_rows, b.second - b.first);
      int *rel = (int *)dalloc((max_rows + 1) * 4);
      size_t tb_max = 0;
      for (auto &b : batches) {
        size_t tb = 0;
        const int nitems = (int)(h_off[b.second] - h_off[b.first]);
        const int nseg = (int)(b.second - b.first);
        CK(cub::DeviceSegmentedSort::StableSortPairs(nullptr, tb, kin, kout, vout, vout, nitems, nseg, rel, rel + 1));
        tb_max = std::max(tb_max, tb);
      }
      void *temp = dalloc(tb_max);
      for (auto &b : batches) {
        const unsigned long long base = h_off[b.first];
        const int nitems = (int)(h_off[b.second] - base);
        const int nseg = (int)(b.second - b.first);
        if (nitems == 0) continue;
        uint32_t *vals = d_adj + base;
        hubkey_kernel<<<4096, 256>>>(vals, d_kdeg, (unsigned long long)nitems, kin);
        rel_offsets_kernel<<<(nseg + 256) / 256, 256>>>(d_off, b.first, (uint32_t)nseg, rel);
        CK(cudaGetLastError());
        size_t tb = tb_max;
        CK(cub::DeviceSegmentedSort::StableSortPairs(temp, tb, kin, kout, vals, vout, nitems, nseg, rel, rel + 1));
        CK(cudaMemcpy(vals, vout, (size_t)nitems * 4, cudaMemcpyDeviceToDevice));
      }
      CK(cudaDeviceSynchronize());
    } catch (...) {
      for (void *p : tmp) cudaFree(p);
      throw;
    }
    for (void *p : tmp) cudaFree(p);
  });
}

extern "C" int ibfs_graph_info(const ibfs_graph *g, uint32_t *nv, uint64_t *ne, uint32_t *max_degree,
                               int *device) {
  return guarded([&] {
    if (!g) fail(IBFS_E_INVALID, "graph is NULL");
    if (nv) *nv = g->nv;
    if (ne) *ne = g->ne;
    if (max_degree) *max_degree = g->max_deg;
    if (device) *device = g->device;
  });
}

extern "C" int ibfs_graph_export_csr(const ibfs_graph *g, uint64_t *offsets, uint32_t *adj) {
  return guarded([&] {
    if (!g || !offsets || (g->ne && !adj)) fail(IBFS_E_INVALID, "NULL argument");
    DeviceScope ds(g->device);
    // back to caller ids: offsets[v] = compacted offset of the first vertex of degree > 0
    // at or after v (isolated rows are empty); adjacency ids through the inverse rank map
    std::vector<uint32_t> orig;
    orig.reserve(g->nva);
    for (uint32_t v = 0; v < g->nv; ++v)
      if ((g->h_nzbits[v >> 5] >> (v & 31)) & 1u) orig.push_back(v);
    for (uint32_t v = 0, r = 0; v <= g->nv; ++v) {
      offsets[v] = g->h_off[r];
      if (v < g->nv && ((g->h_nzbits[v >> 5] >> (v & 31)) & 1u)) ++r;
    }
    if (g->ne) {
      CK(cudaMemcpy(adj, g->d_adj, g->ne * 4, cudaMemcpyDeviceToHost));
      for (uint64_t i = 0; i < g->ne; ++i) adj[i] = orig[adj[i]];
    }
  });
}

extern "C" void ibfs_free(ibfs_graph *g) { graph_release(g); }

extern "C" int ibfs_set_allocator(void *(*alloc)(size_t, int, void *), void (*release)(void *, int, void *),
                                  void *ctx) {
  return guarded([&] {
    if ((alloc == nullptr) != (release == nullptr)) fail(IBFS_E_INVALID, "alloc and release must both be set or both NULL");
    std::lock_guard<std::mutex> lk(g_alloc_mu);
    g_alloc.alloc = alloc;
    g_alloc.release = release;
    g_alloc.ctx = ctx;
  });
}

// ----------------------------------------------------------------------- planning ----
namespace {
// hub[r] per DESIGN.md reading #16: the neighbour w of sources[r] with deg(w) > q (any
// degree if `uniform`) maximising (deg(w), -w); 0xffffffff if none.  One warp per source.
__global__ void hub_kernel(const unsigned long long *off, const uint32_t *adj, const uint32_t *deg,
                           const uint32_t *src, uint32_t n, uint32_t q, int uniform, uint32_t *hub,
                           uint32_t *sdeg) {
  const int lane = threadIdx.x & 31;
  const uint32_t warps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < n; r += warps) {
    const uint32_t s = src[r];
    if (s == NO_VERTEX) {  // isolated source: no hub, degree 0
      if (lane == 0) { hub[r] = 0xffffffffu; sdeg[r] = 0; }
      continue;
    }
    const unsigned long long e0 = off[s], e1 = off[s + 1];
    unsigned long long best = 0;
    bool have = false;
    for (unsigned long long e = e0 + lane; e < e1; e += 32) {
      const uint32_t w = adj[e];
      const uint32_t dw = deg[w];
      if (uniform || dw > q) {
        const unsigned long long key = ((unsigned long long)dw << 32) | (0xffffffffu - w);
        if (!have || key > best) { best = key; have = true; }
      }
    }
    // warp max over (have, best)
    unsigned long long k = have ? best + 1 : 0;  // +1 keeps "none" = 0 distinct
    for (int o = 16; o > 0; o >>= 1) {
      unsigned long long y = __shfl_xor_sync(FULL, k, o);
      k = y > k ? y : k;
    }
    if (lane == 0) {
      hub[r] = k ? (0xffffffffu - (uint32_t)((k - 1) & 0xffffffffull)) : 0xffffffffu;
      sdeg[r] = deg[s];
    }
  }
}
}  // namespace

extern "C" void ibfs_plan_params_default(ibfs_plan_params *p) {
  if (!p) return;
  std::memset(p, 0, sizeof(*p));
  p->mode = 0;
  p->q = 128;
  p->n_p = 4;
  p->p[0] = 4; p->p[1] = 16; p->p[2] = 64; p->p[3] = 128;
  p->hops = 1;
  p->seed = 3;
}

extern "C" int ibfs_plan_groups(const ibfs_graph *g, const uint32_t *sources, uint32_t n,
                                uint32_t group_bits, const ibfs_plan_params *params, uint32_t *out_perm,
                                uint32_t *out_n_groups) {
  return guarded([&] {
    if (!g) fail(IBFS_E_INVALID, "graph is NULL");
    if (group_bits != 32 && group_bits != 64 && group_bits != 128) fail(IBFS_E_INVALID, "group_bits must be 32, 64 or 128");
    if (n > 0 && (!sources || !out_perm)) fail(IBFS_E_INVALID, "sources/out_perm is NULL");
    ibfs_plan_params pp;
    if (params) pp = *params; else ibfs_plan_params_default(&pp);
    if (pp.mode > 2) fail(IBFS_E_INVALID, "plan mode must be 0, 1 or 2");
    if (pp.mode == 0 && (pp.n_p < 1 || pp.n_p > 8)) fail(IBFS_E_INVALID, "n_p must be 1..8");
    if (pp.mode == 0 && pp.hops != 1 && pp.hops != 2) fail(IBFS_E_INVALID, "hops must be 1 or 2");
    if (out_n_groups) *out_n_groups = (n + group_bits - 1) / group_bits;
    if (n == 0) return;
    std::vector<uint32_t> hsrc(n);
    DeviceScope ds(g->device);
    // device-resident sources: the caller completes the work that wrote them first
    // (include/ibfs.h); a full device sync orders this read after every stream
    if (is_device_ptr(sources)) CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(hsrc.data(), sources, (size_t)n * 4, cudaMemcpyDefault));
    for (uint32_t r = 0; r < n; ++r)
      if (hsrc[r] >= g->nv) fail(IBFS_E_INVALID, "source id >= nv");
    for (uint32_t r = 0; r < n; ++r) hsrc[r] = host_compact_id(g, hsrc[r]);  // planner works on compacted ids
    std::vector<uint32_t> hub(n, 0xffffffffu), sdeg(n, 0), anchor, hubx;
    if (pp.mode == 0) {
      uint32_t *d_src = nullptr, *d_hub = nullptr, *d_sdeg = nullptr;
      CK(cudaMalloc(&d_src, (size_t)n * 4));
      CK(cudaMalloc(&d_hub, (size_t)n * 4));
      CK(cudaMalloc(&d_sdeg, (size_t)n * 4));
      CK(cudaMemcpy(d_src, hsrc.data(), (size_t)n * 4, cudaMemcpyHostToDevice));
      const int uniform = g->max_deg <= pp.q ? 1 : 0;
      uint32_t blocks = std::min<uint32_t>((n + 7) / 8, 65535u);
      hub_kernel<<<blocks, 256>>>(g->d_off, g->d_adj, g->d_deg, d_src, n, pp.q, uniform, d_hub, d_sdeg);
      cudaError_t e = cudaGetLastError();
      if (e == cudaSuccess) e = cudaMemcpy(hub.data(), d_hub, (size_t)n * 4, cudaMemcpyDeviceToHost);
      if (e == cudaSuccess) e = cudaMemcpy(sdeg.data(), d_sdeg, (size_t)n * 4, cudaMemcpyDeviceToHost);
      if (e == cudaSuccess && pp.hops == 2) {
        // hub of each source's hub (the same search from the hub vertex); anchor = the
        // larger of the two by (degree desc, id asc)
        std::vector<uint32_t> hv(n), hub2(n, 0xffffffffu);
        // a source without a hub reaches the core through its max-degree neighbour m(r)
        // (any degree, the P:L661 rule): its hub becomes hub(m(r))
        for (uint32_t r = 0; r < n; ++r) hv[r] = (hub[r] == 0xffffffffu && sdeg[r] > 0) ? hsrc[r] : NO_VERTEX;
        e = cudaMemcpy(d_src, hv.data(), (size_t)n * 4, cudaMemcpyHostToDevice);
        if (e == cudaSuccess) {
          hub_kernel<<<blocks, 256>>>(g->d_off, g->d_adj, g->d_deg, d_src, n, pp.q, 1, d_hub, d_sdeg);
          e = cudaGetLastError();
        }
        if (e == cudaSuccess) e = cudaMemcpy(hv.data(), d_hub, (size_t)n * 4, cudaMemcpyDeviceToHost);
        for (uint32_t r = 0; r < n; ++r) if (hv[r] == 0xffffffffu) hv[r] = NO_VERTEX;  // m(r)
        if (e == cudaSuccess) e = cudaMemcpy(d_src, hv.data(), (size_t)n * 4, cudaMemcpyHostToDevice);
        if (e == cudaSuccess) {
          hub_kernel<<<blocks, 256>>>(g->d_off, g->d_adj, g->d_deg, d_src, n, pp.q, uniform, d_hub, d_sdeg);
          e = cudaGetLastError();
        }
        if (e == cudaSuccess) e = cudaMemcpy(hub2.data(), d_hub, (size_t)n * 4, cudaMemcpyDeviceToHost);
        hubx = hub;  // step 3 buckets by the 1-hop hub; the ordering uses the extended one
        for (uint32_t r = 0; r < n; ++r)
          if (hub[r] == 0xffffffffu && sdeg[r] > 0) hubx[r] = hub2[r];  // hub(m(r)) (or none)
        for (uint32_t r = 0; r < n; ++r) hv[r] = hubx[r] == 0xffffffffu ? NO_VERTEX : hubx[r];
        e = cudaMemcpy(d_src, hv.data(), (size_t)n * 4, cudaMemcpyHostToDevice);
        if (e == cudaSuccess) {
          hub_kernel<<<blocks, 256>>>(g->d_off, g->d_adj, g->d_deg, d_src, n, pp.q, uniform, d_hub, d_sdeg);
          e = cudaGetLastError();
        }
        if (e == cudaSuccess) e = cudaMemcpy(hub2.data(), d_hub, (size_t)n * 4, cudaMemcpyDeviceToHost);
        anchor.assign(n, 0xffffffffu);
        for (uint32_t r = 0; r < n; ++r) {
          uint32_t a = hubx[r];
          const uint32_t b = hub2[r];
          if (a != 0xffffffffu && b != 0xffffffffu) {
            const uint64_t da = g->h_off[a + 1] - g->h_off[a], db = g->h_off[b + 1] - g->h_off[b];
            if (db > da || (db == da && b < a)) a = b;
          }
          anchor[r] = a;
        }
      }
      cudaFree(d_src);
      cudaFree(d_hub);
      cudaFree(d_sdeg);
      CK(e);
    }
    auto deg_of = [&](uint32_t x) -> uint64_t { return g->h_off[x + 1] - g->h_off[x]; };
    const bool two = pp.mode == 0 && pp.hops == 2;
    ibfs::plan::make_plan(pp, group_bits, n, hub, sdeg, deg_of, out_perm, two ? &anchor : nullptr,
                          two ? &hubx : nullptr);
  });
}

// ---------------------------------------------------------------------- traversal ----
extern "C" void ibfs_run_opts_default(ibfs_run_opts *o) {
  if (!o) return;
  std::memset(o, 0, sizeof(*o));
  o->direction = IBFS_DIR_AUTO;
  o->bu_from = 2;
  o->alpha = 3.0f;  // profiles/r02/direction: c3 +4 %, c4 +3 %, c5 +0.5 % over 4
  o->beta = 24.0f;
  o->split = IBFS_SPLIT_AUTO;
  o->split_mod = 2;
  o->split_div = 512.0f;  // A/B sweep, profiles/r02/split_div.md
}

namespace {

constexpr int LEVELS_PER_CHECK = 4;  // levels per polled chunk; two chunks stay queued ahead

// cuTensorMapEncodeTiled through the runtime's driver entry point (no libcuda link).
PFN_cuTensorMapEncodeTiled_v12000 tensor_map_encoder() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    cudaGetLastError();
  });
  return fn;
}

// Depth rows through 2-D TMA tensor stores (depth_tma_kernel) unless IBFS_DEPTH_TMA=0
// (A/B runs) or the rows break the tensor map rules (row pitch nv and base 16-byte aligned).
// Bottom-up frontier-bitmap probes: IBFS_BU_PROBE = 0 never, 1 when the frontier is small
// (default), 2 always (A/B runs; results never change).
uint32_t bu_probe_mode() {
  static const uint32_t m = [] {
    const char *e = std::getenv("IBFS_BU_PROBE");
    return (e && e[0] >= '0' && e[0] <= '2') ? (uint32_t)(e[0] - '0') : 1u;
  }();
  return m;
}

bool env_flag(const char *name, bool dflt) {
  const char *e = std::getenv(name);
  return e ? e[0] == '1' : dflt;
}

// Clean ring unless IBFS_CLEAN_RING=0 (A/B runs: the commits clear the next
// slot every level, as in round 1).  IBFS_CHECK_RING=1 (tests) verifies after every call
// that the ring is all zero again and fails with IBFS_E_CUDA otherwise.
bool clean_ring_enabled() {
  static const bool on = [] {
    const char *e = std::getenv("IBFS_CLEAN_RING");
    return !(e && e[0] == '0');
  }();
  return on;
}
// IBFS_FUSED_CLEAN=1 (A/B runs): the depth kernel's consumers zero the runs they read
// (W = 128) instead of ring_clean_kernel.  Measured (profiles/r02/clean_ring/): c5 depth
// flush +20.5 ms per 8 steps against 11.5 ms for the separate pass, c3 -1 ms: off by default.
bool fused_clean_enabled() {
  static const bool on = [] {
    const char *e = std::getenv("IBFS_FUSED_CLEAN");
    return e && e[0] == '1';
  }();
  return on;
}
bool ms_clean_enabled() {
  static const bool on = env_flag("IBFS_MS_CLEAN", true);
  return on;
}
bool check_ring_enabled() {
  const char *e = std::getenv("IBFS_CHECK_RING");
  return e && e[0] == '1';
}

// IBFS_SPLIT_REL=x (A/B runs): in a split bottom-up level, also expand top-down every
// instance whose sampled frontier edge count is below 1/x of the group's largest (0 = off).
float split_rel_default() {
  static const float v = [] {
    const char *e = std::getenv("IBFS_SPLIT_REL");
    return e ? (float)std::atof(e) : 0.f;
  }();
  return v;
}

bool depth_tma_enabled() {
  static const bool on = [] {
    const char *e = std::getenv("IBFS_DEPTH_TMA");
    return !(e && e[0] == '0');
  }();
  return on;
}

// Tensor map of a batch's rows: int8 [rows][nv] at `out`, boxes of DV columns x W rows.
bool make_rows_tensor_map(CUtensorMap *m, int8_t *out, uint32_t nv, uint32_t rows, uint32_t W) {
  PFN_cuTensorMapEncodeTiled_v12000 enc = tensor_map_encoder();
  if (!enc || (nv % 16) != 0 || ((uintptr_t)out % 16) != 0 || rows == 0) return false;
  cuuint64_t dims[2] = {(cuuint64_t)nv, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)nv};
  cuuint32_t box[2] = {(cuuint32_t)DV, (cuuint32_t)W};
  cuuint32_t estr[2] = {1, 1};
  return enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, out, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
             CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
             CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Per-thread, per-device cache of CUDA events and a pinned host word buffer: creating
// them per call (cudaEventCreate, cudaMallocHost) costs far more than a small level.
struct DevCache {
  std::vector<cudaEvent_t> timed, untimed;
  void *pinned = nullptr;
  void *stage = nullptr;  // pinned host staging of per-batch statistics (grown on demand)
  size_t stage_bytes = 0;
  void *host_stage(size_t bytes) {
    if (bytes > stage_bytes) {
      if (stage) cudaFreeHost(stage);
      stage = nullptr;
      stage_bytes = 0;
      CK(cudaMallocHost(&stage, bytes));
      stage_bytes = bytes;
    }
    return stage;
  }
};
struct ThreadCache {
  std::vector<std::pair<int, DevCache>> devs;
  ~ThreadCache() {
    for (auto &d : devs) {
      for (auto e : d.second.timed) cudaEventDestroy(e);
      for (auto e : d.second.untimed) cudaEventDestroy(e);
      if (d.second.pinned) cudaFreeHost(d.second.pinned);
      if (d.second.stage) cudaFreeHost(d.second.stage);
    }
  }
  DevCache &get(int dev) {
    for (auto &d : devs)
      if (d.first == dev) return d.second;
    devs.push_back({dev, DevCache{}});
    return devs.back().second;
  }
};
thread_local ThreadCache t_cache;

struct EventTimer {
  std::vector<cudaEvent_t> &pool;
  bool timing;
  size_t used = 0;
  EventTimer(DevCache &dc, bool timed) : pool(timed ? dc.timed : dc.untimed), timing(timed) {}
  cudaEvent_t next() {
    if (used == pool.size()) {
      cudaEvent_t e;
      CK(cudaEventCreateWithFlags(&e, timing ? cudaEventDefault : cudaEventDisableTiming));
      pool.push_back(e);
    }
    return pool[used++];
  }
};

using HostClock = std::chrono::steady_clock;
double ms_since(HostClock::time_point t0) {
  return std::chrono::duration<double, std::milli>(HostClock::now() - t0).count();
}
// blocks on an event, adding the blocked time to *wait_ms
void wait_event(cudaEvent_t e, double *wait_ms) {
  const auto t = HostClock::now();
  CK(cudaEventSynchronize(e));
  *wait_ms += ms_since(t);
}

template <typename T>
void run_typed(const ibfs_graph *g, const uint32_t *sources, uint32_t n,
               int8_t *out_depths, const ibfs_run_opts &o, ibfs_stats *stats, HostClock::time_point t_entry) {
  constexpr int W = WordBits<T>::value;
  constexpr size_t B = sizeof(T);
  cudaStream_t stream = (cudaStream_t)o.cuda_stream;
  const uint32_t nv = g->nv, nva = g->nva;
  const uint32_t n_groups = (n + W - 1) / W;
  const bool out_dev = is_device_ptr(out_depths);
  const bool out_host = out_depths && !out_dev;

  // groups per launch batch
  uint32_t G = o.groups_in_flight;
  if (G == 0) {
    // auto: ~32 M status words per launch batch and at least 4 groups -- several groups
    // share every level launch (a9), so one group's small levels overlap another's large
    // ones and the host polls once per batch; the memory budget below caps it
    uint64_t want = std::max<uint64_t>((32ull << 20) / std::max<uint32_t>(nva, 1) + 1, 4);
    G = (uint32_t)std::min<uint64_t>(want, MAX_G);
  }
  G = std::max<uint32_t>(1, std::min<uint32_t>({G, (uint32_t)MAX_G, n_groups}));
  const size_t gstride = ((size_t)nva + 16) & ~(size_t)15;
  const size_t rows_bytes_per_group = (size_t)W * nv;
  const size_t total_b = g->total_mem;
  // memory: visited + R snapshot slots per group (+ device rows if the caller's buffer
  // is not on the device); R >= 4, up to one slot per level when memory allows
  auto need = [&](uint32_t gg, uint32_t r) {
    return gg * ((1 + r) * gstride * B + 8 * (size_t)nva + (out_dev ? 0 : rows_bytes_per_group)) + (size_t)n * 28;
  };
  // The budget depends on the device size only (not on the momentary free memory), so
  // repeated calls request identical scratch and the stream-ordered pool reuses it.
  const size_t budget = total_b / 100 * 35;
  while (G > 1 && need(G, 4) > budget) G = (G + 1) / 2;
  uint32_t R = 4;
  while (R < 24 && need(G, R + 1) <= budget) ++R;  // > R-2 levels: flushed ring rounds

  Scratch sc(g->device, stream, const_cast<ScratchCache *>(&g->scratch));
  uint32_t *d_src = sc.get<uint32_t>(n);
  CK(cudaMemcpyAsync(d_src, sources, (size_t)n * 4, cudaMemcpyDefault, stream));
  uint32_t *d_csrc = sc.get<uint32_t>(n);
  compact_sources_kernel<<<(n + 255) / 256, 256, 0, stream>>>(d_src, n, g->d_tbase, g->d_nzbits, d_csrc);
  CK(cudaGetLastError());
  // clean ring: visited too is all zero between calls (ms_kernel zeroes each word after
  // reading it), so init only sets the sources
  const bool clean_ring = clean_ring_enabled();
  int vis_idx = -1;
  T *visited = clean_ring ? sc.get_zeroed<T>(G * gstride, &vis_idx) : sc.get<T>(G * gstride);
  // clean ring: all slots zero at batch start, zeroed again after the depth
  // rows are written; a ring the previous call did not leave zero is cleared once here
  int ring_idx = -1;
  T *ring = clean_ring ? sc.get_zeroed<T>((size_t)R * G * gstride, &ring_idx) : sc.get<T>((size_t)R * G * gstride);
  uint32_t *tdq = sc.get<uint32_t>((size_t)G * std::max<uint32_t>(nva, 1));
  uint32_t *buq = sc.get<uint32_t>((size_t)G * std::max<uint32_t>(nva, 1));
  const uint32_t nchunk32 = (nva + 31) / 32;
  uint8_t *dirty = sc.get<uint8_t>((size_t)G * std::max<uint32_t>(nchunk32, 1));
  uint32_t *fbits = sc.get<uint32_t>((size_t)G * std::max<uint32_t>(nchunk32, 1));
  const uint32_t late_cap = o.late_cap ? o.late_cap : nva / 32 + 1024;  // new vertices of sparse levels (per group)
  unsigned long long *late = sc.get<unsigned long long>((size_t)G * late_cap);
  uint32_t *late_n = sc.get<uint32_t>(G);
  const uint32_t chq_stride = std::max<uint32_t>(std::max(g->n_chunks, g->n_rchunks), 1);
  uint32_t *chq = sc.get<uint32_t>((size_t)G * 2 * chq_stride);
  GroupCtrl<T> *ctrl = sc.get<GroupCtrl<T>>(G);
  LevelStat *lstat = sc.get<LevelStat>((size_t)G * MAXL);
  uint32_t *work_ctr = sc.get<uint32_t>(MAXL);
  uint32_t *flags = sc.get<uint32_t>(4);  // batch_done, range_err, grid barrier (count, generation)
  unsigned long long *tstamp = sc.get<unsigned long long>((size_t)MAXL * 3);

  unsigned long long *d_m = sc.get<unsigned long long>((size_t)G * W);
  unsigned long long *d_dig = sc.get<unsigned long long>((size_t)G * W);
  int8_t *staging = out_dev ? nullptr : sc.get<int8_t>((size_t)G * rows_bytes_per_group);
  CK(cudaMemsetAsync(flags, 0, 16, stream));

  DevCache &dc = t_cache.get(g->device);
  if (!dc.pinned) CK(cudaMallocHost(&dc.pinned, 4096));
  volatile uint32_t *h_done = (volatile uint32_t *)dc.pinned;  // [0..255] done slots, [256] range
  // statistics staging in pinned host memory: level stats [G][MAXL], stamps [MAXL][3],
  // m_s and digests [G*W] each (only the levels a batch ran are copied)
  const size_t st_lstat = (size_t)G * MAXL * sizeof(LevelStat), st_ts = (size_t)MAXL * 3 * 8,
               st_m = (size_t)G * W * 8;
  // two slots: batch b's statistics are copied into slot b % 2 and read on the host while
  // batch b + 1 runs (no device idle between the batches of a call)
  const size_t st_slot = ((st_lstat + st_ts + 2 * st_m + 16) + 255) & ~(size_t)255;
  unsigned char *hst = (unsigned char *)dc.host_stage(2 * st_slot);
  struct Slot {
    LevelStat *lstat;
    unsigned long long *ts, *m, *dig;
    uint32_t *range;
  } slots[2];
  for (int k = 0; k < 2; ++k) {
    unsigned char *b = hst + k * st_slot;
    slots[k].lstat = (LevelStat *)b;
    slots[k].ts = (unsigned long long *)(b + st_lstat);
    slots[k].m = (unsigned long long *)(b + st_lstat + st_ts);
    slots[k].dig = slots[k].m + (size_t)G * W;
    slots[k].range = (uint32_t *)(slots[k].dig + (size_t)G * W);
  }

  BatchArgs<T> a{};
  a.off = g->d_off;
  a.adj = g->d_adj;
  a.deg = g->d_deg;
  a.directed = g->directed ? 1u : 0u;
  a.roff = g->directed ? g->d_roff : g->d_off;
  a.radj = g->directed ? g->d_radj : g->d_adj;
  a.rdeg = g->directed ? g->d_rdeg : g->d_deg;
  a.tbase = g->d_tbase;
  a.nzbits = g->d_nzbits;
  a.nv = nv;
  a.nva = nva;
  a.gstride = gstride;
  a.visited = visited;
  a.ring = ring;
  a.R = (int)R;
  a.gcap = (int)G;
  a.ctrl = ctrl;
  a.lstat = lstat;
  a.work_ctr = work_ctr;
  a.batch_done = flags;
  a.range_err = flags + 1;
  a.gbar = flags + 2;
  a.tstamp = tstamp;
  a.n_total = n;
  a.chunks = g->d_chunks;
  a.n_chunks = g->n_chunks;
  a.hub_vtx = g->d_hub_vtx;
  a.hub_chunk0 = g->d_hub_chunk0;
  a.n_hubs = g->n_hubs;
  a.rchunks = g->directed ? g->d_rchunks : g->d_chunks;
  a.n_rchunks = g->directed ? g->n_rchunks : g->n_chunks;
  a.rhub_vtx = g->directed ? g->d_rhub_vtx : g->d_hub_vtx;
  a.rhub_chunk0 = g->directed ? g->d_rhub_chunk0 : g->d_hub_chunk0;
  a.n_rhubs = g->directed ? g->n_rhubs : g->n_hubs;
  a.chq_stride = chq_stride;
  a.chq = chq;
  a.tdq = tdq;
  a.buq = buq;
  a.dirty = dirty;
  a.fbits = fbits;
  a.nchunk32 = nchunk32;
  a.late = late;
  a.late_n = late_n;
  a.late_cap = late_cap;
  a.clean_ring = clean_ring ? 1u : 0u;
  a.n_iso = nv - nva;
  a.pol.mode = o.direction;
  a.pol.bu_from = o.bu_from;
  a.pol.alpha = o.alpha;
  a.pol.beta = o.beta;
  a.pol.nv_active = g->nv_active;
  a.pol.ne = g->ne;
  a.pol.split = o.split;
  a.pol.split_mod = std::max<uint32_t>(1, o.split_mod);
  a.pol.split_div = o.split_div;
  a.pol.max_depth = o.max_depth;
  a.pol.bu_probe = bu_probe_mode();
  a.pol.split_rel = split_rel_default();
  {  // A/B: profiles/r02/td_scheck (1: c5 +2 %)
    const char *e = std::getenv("IBFS_TD_SCHECK");
    a.pol.td_scheck = (e && e[0] >= '0' && e[0] <= '2') ? (uint32_t)(e[0] - '0') : 1u;
  }
  a.pol.sched_len = std::min<uint32_t>(o.schedule_len, MAXL);
  for (uint32_t i = 0; i < a.pol.sched_len; ++i) a.pol.sched[i] = (o.schedule[i] == 'B' || o.schedule[i] == 1) ? 1 : 0;
  uint32_t first_dir = 0;
  if (o.direction == IBFS_DIR_BU_FROM) first_dir = o.bu_from <= 1 ? 1 : 0;
  if (o.direction == IBFS_DIR_SCHEDULE && a.pol.sched_len > 0) first_dir = a.pol.sched[0];

  const int level_grid = g->num_sms * g->level_blocks_per_sm[W == 32 ? 0 : (W == 64 ? 1 : 2)];
  EventTimer timer(dc, true), chk(dc, false);
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> win, klev, kinit, kdep, kfin, kms, kcopy, kcl;
  ibfs_stats st{};
  uint64_t launches = 0;
  bool range_error = false;
  std::vector<ibfs_level_stats> per_level(MAXL);

  struct Pending {
    bool valid = false;
    uint32_t gb0 = 0, Gb = 0, rows = 0;
    int level = 0, slot = 0;
    int fused_from = 1 << 30;  // levels >= this were zeroed by the depth kernel (fused clean)
    int ms_from = 1 << 30;     // levels >= this were zeroed by the m_s pass
    cudaEvent_t done = nullptr;
  } pend;
  // host side of a finished batch: per-source outputs, level records, byte models, times
  double wait_ms = 0, setup_ms = -1;
  auto harvest = [&](const Pending &pb) {
    wait_event(pb.done, &wait_ms);
    const Slot &sl = slots[pb.slot];
    const uint32_t gb0 = pb.gb0, Gb = pb.Gb, rows_in_batch = pb.rows;
    const int level = pb.level;
    const int lrows = std::min(level + 1, MAXL);
    const LevelStat *h_lstat = sl.lstat;
    const unsigned long long *h_ts = sl.ts, *h_mp = sl.m, *h_digp = sl.dig;
    if (*sl.range) range_error = true;
    // accumulate per-source outputs and statistics
    for (uint32_t r = 0; r < rows_in_batch; ++r) {
      st.edges_traversed += h_mp[r];
      if (stats && stats->per_source_m) stats->per_source_m[(size_t)gb0 * W + r] = h_mp[r];
      if (stats && stats->per_source_digest) stats->per_source_digest[(size_t)gb0 * W + r] = h_digp[r];
    }
    for (uint32_t gi = 0; gi < Gb; ++gi) {
      for (int l = 1; l < lrows; ++l) {
        const LevelStat &L = h_lstat[(size_t)gi * MAXL + l];
        if (L.dir == 0) continue;
        ibfs_level_stats &P = per_level[l - 1];
        const bool td = L.dir == 1;
        st.max_levels = std::max<uint32_t>(st.max_levels, (uint32_t)l);
        if (td) { P.td_groups++; P.jfq_td += L.jfq; P.fq_td += L.fq; st.levels_td++; st.sd_fq_td += L.fq; st.sd_jfq_td += L.jfq; }
        else { P.bu_groups++; P.jfq_bu += L.jfq; P.fq_bu += L.fq; st.levels_bu++; st.sd_fq_bu += L.fq; st.sd_jfq_bu += L.jfq; }
        P.inspected += L.insp;
        P.new_pairs += L.newp;
        P.gathered += L.gath;
        st.words_gathered += L.gath;
        st.edges_inspected += L.insp;
        // DESIGN.md §5 byte model (SURVEY.md §8(d) "Algorithmic bytes")
        // expand: per queued frontier its row start and word; per inspection the adjacency
        // entry (4 B); the neighbour's word (B) only when it is gathered -- a bottom-up
        // frontier-bitmap hit or a top-down pre-check; per S_l write one
        // word; a bottom-up level reads the group's frontier bitmap (nva / 8 B) once.
        // commit (§8(d) dense scan): S_l and visited read, the next slot cleared, visited
        // written where new, the frontier bitmap written (nva / 8 B).
        uint64_t eb = (8 + B) * L.proc + 4 * L.insp + B * L.gath + B * L.writes + (L.dir == 2 ? (uint64_t)nchunk32 * 4 : 0);
        uint64_t cb = (uint64_t)nva * ((clean_ring ? 2 : 3) * B) + B * L.nf + (uint64_t)nchunk32 * 4;
        st.expand_bytes += eb;
        st.commit_bytes += cb;
        // what the commit streams: dense -- S_l, visited, the cleared slot, degrees (and
        // in-degrees), the chunk map; sparse -- the chunk map, the marked chunks (at most
        // one per write) and the cleared slot
        const uint64_t degb = g->directed ? 8 : 4;
        if (L.flags & 2u) {
          const uint64_t chunks = std::min<uint64_t>(L.writes, nchunk32);
          st.commit_bytes_moved += nchunk32 * 5ull + chunks * 32 * (2 * B + degb) + (clean_ring ? 0 : (uint64_t)nva * B) + B * L.nf;
        } else {
          st.commit_bytes_moved += (uint64_t)nva * ((clean_ring ? 2 : 3) * B + degb) + nchunk32 * 5ull + B * L.nf;
        }
        // clean ring: a loaded level's slot is zeroed after the depth pass (B per vertex);
        // a skipped level's late entries are zeroed by the fix-up (B per entry)
        if (clean_ring) {
          if (L.flags & 1u) st.clean_bytes += (uint64_t)L.nf * B;
          else if (l >= pb.fused_from) st.depth_bytes += (uint64_t)nva * B;  // the depth kernel's zero stores
          else if (l >= pb.ms_from) st.ms_bytes += (uint64_t)nva * B;        // the m_s pass's zero stores
          else st.clean_bytes += (uint64_t)nva * B;
        }
        // depth kernel: a loaded level's snapshot is read once; a skipped level's new
        // vertices (<= nf) are read back from the late list (entry + word) instead
        if (L.flags & 1u) st.depth_bytes += (uint64_t)L.nf * (B + 8);
        else st.depth_bytes += (uint64_t)nva * B;
      }
    }
    for (int l = 1; l < level; ++l)  // launches of levels 1..level-1 were queued
      if (h_ts[(size_t)l * 3] != ~0ull) st.level_launches_live++;
    // phase times of each level kernel from its in-kernel globaltimer stamps: [first CTA
    // start, grid barrier, last CTA end]; the commit part belongs to level l-1
    for (int l = 1; l < lrows; ++l) {
      const unsigned long long t0 = h_ts[(size_t)l * 3], t1 = h_ts[(size_t)l * 3 + 1], t2 = h_ts[(size_t)l * 3 + 2];
      if (t0 == ~0ull || t1 < t0 || t2 < t1) continue;
      const double cms = (t1 - t0) * 1e-6, ems = (t2 - t1) * 1e-6;
      st.expand_ms += ems;
      per_level[l - 1].expand_ms += ems;
      if (l > 1) {
        st.commit_ms += cms;
        per_level[l - 2].commit_ms += cms;
      }
    }
    for (int l = 1; l + 1 < lrows; ++l) {  // idle between level l's last CTA and level l+1's first
      const unsigned long long e = h_ts[(size_t)l * 3 + 2], b = h_ts[(size_t)(l + 1) * 3];
      if (e && b != ~0ull && b > e) st.level_gap_ms += (b - e) * 1e-6;
    }
  };
  int batch_no = 0;
  for (uint32_t gb0 = 0; gb0 < n_groups; gb0 += G, ++batch_no) {
    const uint32_t Gb = std::min(G, n_groups - gb0);
    const Slot &sl = slots[batch_no & 1];
    a.G = (int)Gb;
    a.group0 = gb0;
    a.src = d_src + (size_t)gb0 * W;
    a.csrc = d_csrc + (size_t)gb0 * W;
    a.out = out_dev ? out_depths + (size_t)gb0 * rows_bytes_per_group : staging;
    const uint32_t rows_in_batch = std::min<uint32_t>(Gb * W, n - gb0 * W);
    CK(cudaMemsetAsync(flags, 0, 4, stream));
    CK(cudaMemsetAsync(late_n, 0, (size_t)G * 4, stream));
    CK(cudaMemsetAsync(d_m, 0, (size_t)G * W * 8, stream));  // m_s accumulates in ms_kernel
    cudaEvent_t w0 = timer.next(), w1 = timer.next();
    CK(cudaEventRecord(w0, stream));
    {
      cudaEvent_t i0 = nullptr, i1 = nullptr;
      if (o.timing) { i0 = timer.next(); i1 = timer.next(); CK(cudaEventRecord(i0, stream)); }
      uint32_t bx = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(((uint64_t)nva + BLOCK - 1) / BLOCK, std::max<uint32_t>(1, 2048 / Gb)));
      if (setup_ms < 0) setup_ms = ms_since(t_entry);
      init_ctrl_kernel<T><<<Gb, 128, 0, stream>>>(a, first_dir);
      init_state_kernel<T><<<dim3(bx, Gb), BLOCK, 0, stream>>>(a, first_dir);
      init_sources_kernel<T><<<Gb, 128, 0, stream>>>(a, first_dir);
      CK(cudaGetLastError());
      launches += 3;
      st.init_launches += 3;
      st.init_bytes += (uint64_t)Gb * (clean_ring ? (uint64_t)nchunk32 * 5 : 3 * (uint64_t)nva * B);
      if (o.timing) { CK(cudaEventRecord(i1, stream)); kinit.push_back({i0, i1}); }
    }
    // depth flush: rows from snapshots [l0, l1] (first flush writes every byte)
    int flushed = -1;  // levels <= flushed are already in the rows
    int fused_from = 1 << 30;
    int ms_from = 1 << 30;
    bool batch_iso = false;  // a source of this batch is isolated (its own zero is a fix-up)
    for (uint32_t r = 0; r < rows_in_batch; ++r) {
      const uint32_t v = sources[(size_t)gb0 * W + r];
      batch_iso |= ((g->h_nzbits[v >> 5] >> (v & 31)) & 1u) == 0;
    }
    auto flush = [&](int l1, bool final_flush) {
      cudaEvent_t d0 = nullptr, d1 = nullptr, m0 = nullptr, m1 = nullptr;
      if (o.timing) { d0 = timer.next(); d1 = timer.next(); CK(cudaEventRecord(d0, stream)); }
      const uint32_t bx = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(((uint64_t)nv + DV - 1) / DV,
                                                                         std::max<uint64_t>(1, (uint64_t)g->num_sms * g->depth_blocks_per_sm[W == 32 ? 0 : (W == 64 ? 1 : 2)] / Gb)));
      const int first = flushed < 0 ? 1 : 0;
      CUtensorMap tmap;
      bool fused_clean = false;  // the depth kernel zeroes the runs it loaded (clean ring, W = 128)
      bool clean_in_ms = false;  // the m_s pass zeroed them
      if (first && depth_tma_enabled() && make_rows_tensor_map(&tmap, a.out, nv, rows_in_batch, W)) {
        fused_clean = clean_ring && B == 16 && fused_clean_enabled();
        if (fused_clean) fused_from = std::min(fused_from, flushed + 1);
        const uint32_t bt = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(((uint64_t)nv + DV - 1) / DV,
                                                                           std::max<uint64_t>(1, (uint64_t)g->num_sms * g->dtma_blocks_per_sm[W == 32 ? 0 : (W == 64 ? 1 : 2)] / Gb)));
        depth_tma_kernel<T><<<dim3(bt, Gb), DTHREADS + 32, depth_tma_smem_bytes<T>(), stream>>>(tmap, a, flushed + 1, l1, fused_clean ? 1 : 0);
      } else {
        depth_kernel<T><<<dim3(bx, Gb), DTHREADS + 32, depth_smem_bytes<T>(), stream>>>(a, flushed + 1, l1, first);
      }
      launches++;
      st.depth_launches++;
      // rows: each (instance, vertex) byte once per batch (§8(d) "i·|V| bytes"); the
      // snapshot reads are counted per group from the level records after the batch
      if (first) st.depth_rows_bytes += (uint64_t)rows_in_batch * nv;
      if (o.timing) { CK(cudaEventRecord(d1, stream)); kdep.push_back({d0, d1}); m0 = timer.next(); m1 = timer.next(); CK(cudaEventRecord(m0, stream)); }
      late_fix_kernel<T><<<dim3(std::min<uint32_t>((late_cap + 255) / 256, 64), Gb), 256, 0, stream>>>(a, flushed + 1, l1);
      launches++;
      st.ms_launches++;
      if (first && batch_iso) {
        iso_fix_kernel<T><<<Gb, 128, 0, stream>>>(a);
        launches++;
        st.ms_launches++;
      }
      if (final_flush) {  // m_s from the final visited words (reading #11)
        const uint32_t mx = (uint32_t)std::max<uint64_t>(
            1, std::min<uint64_t>(((uint64_t)nva + BLOCK - 1) / BLOCK, std::max<uint64_t>(1, (uint64_t)g->num_sms * 4 / Gb)));
        // clean ring: the m_s pass also zeroes this flush's loaded slots (IBFS_MS_CLEAN=0:
        // the separate ring_clean_kernel pass)
        const bool ms_clean = clean_ring && !fused_clean && ms_clean_enabled();
        ms_kernel<T><<<dim3(mx, Gb), BLOCK, 0, stream>>>(a, d_m, ms_clean ? flushed + 1 : 1, ms_clean ? l1 : 0);
        if (ms_clean) {
          clean_in_ms = true;
          ms_from = std::min(ms_from, flushed + 1);
        }
        launches++;
        st.ms_launches++;
        st.ms_bytes += (uint64_t)Gb * nva * ((clean_ring ? 2 * B : B) + 4);  // + the visited words zeroed
      }
      if (o.timing) { CK(cudaEventRecord(m1, stream)); kms.push_back({m0, m1}); }
      if (clean_ring && !fused_clean && !clean_in_ms) {  // the read slots back to zero (after late_fix read the skipped entries)
        cudaEvent_t c0 = nullptr, c1 = nullptr;
        if (o.timing) { c0 = timer.next(); c1 = timer.next(); CK(cudaEventRecord(c0, stream)); }
        const uint32_t cx = (uint32_t)std::max<uint64_t>(
            1, std::min<uint64_t>(((uint64_t)nva * B / 16 + BLOCK) / BLOCK, std::max<uint64_t>(1, (uint64_t)g->num_sms * 8 / Gb)));
        ring_clean_kernel<T><<<dim3(cx, Gb), BLOCK, 0, stream>>>(a, flushed + 1, l1);
        launches++;
        st.clean_launches++;
        if (o.timing) { CK(cudaEventRecord(c1, stream)); kcl.push_back({c0, c1}); }
      }
      flushed = l1;
    };
    int level = 1;
    int chunk = 0;
    cudaEvent_t chk_ev[256];
    chk.used = 0;  // the previous batch's check events have completed
    while (level <= MAXL - 1) {
      const int lend = std::min(level + LEVELS_PER_CHECK, MAXL);
      for (int l = level; l < lend; ++l) {
        // level l's commit (of level l-1) zeroes slot l % R, which held level l-R: flush it
        // first (levels <= l-2 are committed by then)
        if (l - (int)R > flushed) flush(l - 2, false);
        cudaEvent_t e0 = nullptr, e1 = nullptr;
        if (o.timing) { e0 = timer.next(); e1 = timer.next(); CK(cudaEventRecord(e0, stream)); }
        int lv = l;
        void *kargs[] = {(void *)&a, (void *)&lv};
        CK(cudaLaunchCooperativeKernel((const void *)level_kernel<T>, dim3(level_grid), dim3(BLOCK), kargs,
                                       sizeof(TileQueue<T>), stream));
        if (o.timing) {
          CK(cudaEventRecord(e1, stream));
          klev.push_back({e0, e1});
        }
        launches += 1;
        st.level_launches++;
      }
      CK(cudaGetLastError());
      if (chunk >= 256) fail(IBFS_E_CUDA, "level loop overflow");
      CK(cudaMemcpyAsync((void *)(h_done + chunk), flags, 4, cudaMemcpyDeviceToHost, stream));
      cudaEvent_t ce = chk.next();
      chk_ev[chunk] = ce;
      CK(cudaEventRecord(ce, stream));
      ++chunk;
      level = lend;
      if (chunk >= 2) {
        wait_event(chk_ev[chunk - 2], &wait_ms);
        if (h_done[chunk - 2] >= Gb) break;
      }
    }
    flush(level - 1, true);  // the rest (each group stops at its own last level)
    CK(cudaEventRecord(w1, stream));
    win.push_back({w0, w1});
    // range check (a level-128 discovery means a depth > 127)
    CK(cudaMemcpyAsync(sl.range, flags + 1, 4, cudaMemcpyDeviceToHost, stream));
    // finalize: m_s and digests (outside the traversal window)
    cudaEvent_t f0 = timer.next(), f1 = timer.next();
    CK(cudaEventRecord(f0, stream));
    if (stats && stats->per_source_digest) {
      CK(cudaMemsetAsync(d_dig, 0, (size_t)G * W * 8, stream));
      uint32_t bx = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(((uint64_t)nv + BLOCK - 1) / BLOCK, 64));
      digest_kernel<T><<<dim3(bx, Gb * W), BLOCK, 0, stream>>>(a, d_dig);
      launches++;
    }
    CK(cudaGetLastError());
    CK(cudaEventRecord(f1, stream));
    kfin.push_back({f0, f1});
    const int lrows = std::min(level + 1, MAXL);  // levels 0..level-1 ran (and level is a no-op)
    CK(cudaMemcpy2DAsync(sl.lstat, MAXL * sizeof(LevelStat), lstat, MAXL * sizeof(LevelStat),
                         (size_t)lrows * sizeof(LevelStat), Gb, cudaMemcpyDeviceToHost, stream));
    CK(cudaMemcpyAsync(sl.ts, tstamp, (size_t)lrows * 3 * 8, cudaMemcpyDeviceToHost, stream));
    CK(cudaMemcpyAsync(sl.m, d_m, (size_t)Gb * W * 8, cudaMemcpyDeviceToHost, stream));
    if (stats && stats->per_source_digest)
      CK(cudaMemcpyAsync(sl.dig, d_dig, (size_t)Gb * W * 8, cudaMemcpyDeviceToHost, stream));
    if (out_host) {  // rows of a host buffer: D2H from the staging rows (stream-ordered
                     // before the next batch's depth kernel rewrites them)
      cudaEvent_t c0 = timer.next(), c1 = timer.next();
      CK(cudaEventRecord(c0, stream));
      CK(cudaMemcpyAsync(out_depths + (size_t)gb0 * rows_bytes_per_group, staging,
                         (size_t)rows_in_batch * nv, cudaMemcpyDeviceToHost, stream));
      CK(cudaEventRecord(c1, stream));
      kcopy.push_back({c0, c1});
    }
    Pending cur;
    cur.valid = true;
    cur.gb0 = gb0;
    cur.Gb = Gb;
    cur.rows = rows_in_batch;
    cur.level = level;
    cur.fused_from = fused_from;
    cur.ms_from = ms_from;
    cur.slot = batch_no & 1;
    cur.done = timer.next();  // not from `chk`: its events are recycled every batch
    CK(cudaEventRecord(cur.done, stream));
    // the previous batch's statistics, while this one runs; its slot is reused next
    if (pend.valid) harvest(pend);
    pend = cur;
  }
  if (pend.valid) harvest(pend);
  if (range_error) fail(IBFS_E_RANGE, "a depth exceeds 127 (int8 output)");
  // times
  for (auto &p : win) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.traverse_ms += ms; }
  for (auto &p : klev) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.level_ms += ms; }
  for (auto &p : kinit) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.init_ms += ms; }
  for (auto &p : kfin) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.finalize_ms += ms; }
  for (auto &p : kdep) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.depth_ms += ms; }
  for (auto &p : kms) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.ms_ms += ms; }
  for (auto &p : kcopy) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.copyout_ms += ms; }
  for (auto &p : kcl) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.clean_ms += ms; }
  if (clean_ring && check_ring_enabled()) {
    CK(cudaMemsetAsync(flags, 0, 4, stream));
    const size_t n16 = (size_t)R * G * gstride * B / 16, v16 = (size_t)G * gstride * B / 16;
    ring_check_kernel<<<(uint32_t)std::min<size_t>((n16 + 255) / 256, 4096), 256, 0, stream>>>(
        reinterpret_cast<const uint4 *>(ring), n16, flags);
    ring_check_kernel<<<(uint32_t)std::min<size_t>((v16 + 255) / 256, 4096), 256, 0, stream>>>(
        reinterpret_cast<const uint4 *>(visited), v16, flags);
    uint32_t bad = 0;
    CK(cudaMemcpyAsync(&bad, flags, 4, cudaMemcpyDeviceToHost, stream));
    CK(cudaStreamSynchronize(stream));
    if (bad) fail(IBFS_E_CUDA, "IBFS_CHECK_RING: a ring slot or visited word is not zero after the call");
  }
  if (clean_ring) {  // every batch's clean-up is complete (harvest waited)
    sc.mark_zero(ring_idx);
    sc.mark_zero(vis_idx);
  }
  st.depth_bytes += st.depth_rows_bytes;
  st.n_groups = n_groups;
  st.n_launches = launches;
  st.bytes_algorithmic = st.expand_bytes + st.commit_bytes + st.init_bytes + st.depth_bytes + st.ms_bytes + st.clean_bytes;
  st.host_setup_ms = setup_ms;
  st.host_wait_ms = wait_ms;
  st.host_total_ms = ms_since(t_entry);
  if (stats) {
    st.per_source_m = stats->per_source_m;
    st.per_source_digest = stats->per_source_digest;
    st.level_cap = stats->level_cap;
    st.per_level = stats->per_level;
    if (st.per_level)
      for (uint32_t i = 0; i < st.level_cap; ++i) st.per_level[i] = i < (uint32_t)MAXL ? per_level[i] : ibfs_level_stats{};
    *stats = st;
  }
}


// ---- the byte-JSA joint engine (ablation rung "Joint", joint.cuh) ----------------------
// One group at a time, host-driven levels (a JFQ scan, then the expand); the same
// direction policy as the bitwise engine, decided on the host from the JFQ counters.
void run_joint(const ibfs_graph *g, const uint32_t *sources, const uint32_t *csources, uint32_t n, uint32_t W,
               int8_t *out_depths, const ibfs_run_opts &o, ibfs_stats *stats) {
  using namespace joint;
  cudaStream_t stream = (cudaStream_t)o.cuda_stream;
  const uint32_t nv = g->nv, nva = g->nva;
  const uint32_t n_groups = (n + W - 1) / W;
  const bool out_dev = is_device_ptr(out_depths);
  const bool out_host = out_depths && !out_dev;
  Scratch sc(g->device, stream);
  uint8_t *jsa = sc.get<uint8_t>((size_t)std::max<uint32_t>(nva, 1) * W);
  uint32_t *jfq = sc.get<uint32_t>(std::max<uint32_t>(nva, 1));
  unsigned long long *ctr = sc.get<unsigned long long>(4);
  uint32_t *newcnt = sc.get<uint32_t>(W);
  uint32_t *d_csrc = sc.get<uint32_t>(W);
  unsigned long long *d_m = sc.get<unsigned long long>(W);
  unsigned long long *d_dig = sc.get<unsigned long long>(W);
  int8_t *staging = out_dev ? nullptr : sc.get<int8_t>((size_t)W * nv);
  DevCache &dc = t_cache.get(g->device);
  EventTimer timer(dc, true);
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> win;
  std::vector<ibfs_level_stats> per_level(MAXL);
  ibfs_stats st{};
  uint64_t launches = 0;
  bool range_error = false;
  const int grid = g->num_sms * 8;
  JointArgs a{};
  a.off = g->d_off;
  a.adj = g->d_adj;
  a.roff = g->directed ? g->d_roff : g->d_off;
  a.radj = g->directed ? g->d_radj : g->d_adj;
  a.deg = g->d_deg;
  a.nva = nva;
  a.W = (int)W;
  a.jsa = jsa;
  a.jfq = jfq;
  a.ctr = ctr;
  a.newcnt = newcnt;
  std::vector<uint32_t> h_new(W);
  std::vector<unsigned long long> h_m(W), h_dig(W);
  for (uint32_t gi = 0; gi < n_groups; ++gi) {
    const uint32_t rows = std::min<uint32_t>(W, n - gi * W);
    int8_t *out = out_dev ? out_depths + (size_t)gi * W * nv : staging;
    uint32_t act[4] = {0, 0, 0, 0};
    for (uint32_t j = 0; j < rows; ++j)
      if (csources[(size_t)gi * W + j] != NO_VERTEX) act[j >> 5] |= 1u << (j & 31);
    cudaEvent_t w0 = timer.next(), w1 = timer.next();
    CK(cudaEventRecord(w0, stream));
    CK(cudaMemsetAsync(jsa, 0xff, (size_t)nva * W, stream));
    CK(cudaMemcpyAsync(d_csrc, csources + (size_t)gi * W, rows * 4, cudaMemcpyHostToDevice, stream));
    jsa_sources<<<1, W, 0, stream>>>(a, d_csrc, (int)rows);
    launches++;
    uint32_t dir = 0;  // direction of the level about to run: 0 TD, 1 BU
    if (o.direction == IBFS_DIR_BU_FROM) dir = o.bu_from <= 1 ? 1 : 0;
    if (o.direction == IBFS_DIR_SCHEDULE && o.schedule_len > 0) dir = (o.schedule[0] == 'B' || o.schedule[0] == 1);
    for (int level = 1; level < MAXL; ++level) {
      if ((act[0] | act[1] | act[2] | act[3]) == 0) break;
      std::memcpy(a.act, act, sizeof(act));
      unsigned long long h_ctr[4];
      auto scan = [&](int bu) {
        CK(cudaMemsetAsync(ctr, 0, 32, stream));
        jfq_kernel<<<grid, 256, 0, stream>>>(a, level, bu);
        launches++;
        CK(cudaMemcpyAsync(h_ctr, ctr, 32, cudaMemcpyDeviceToHost, stream));
        CK(cudaStreamSynchronize(stream));
      };
      const bool auto_now = o.direction == IBFS_DIR_AUTO ||
                            (o.direction == IBFS_DIR_SCHEDULE && (uint32_t)level - 1 >= o.schedule_len);
      if (level > 1 && auto_now) {
        // reading #7 on the TD frontier of this level: TD -> BU when m_f * alpha > ne,
        // BU -> TD when n_f * beta < nv_active
        scan(0);
        const double n_f = (double)h_ctr[0], m_f = (double)h_ctr[1];
        dir = dir == 0 ? (m_f > 0 && m_f * o.alpha > (double)g->ne) : !(n_f * o.beta < (double)g->nv_active);
        if (dir) scan(1);
      } else {
        if (o.direction == IBFS_DIR_TD_ONLY) dir = 0;
        if (o.direction == IBFS_DIR_BU_FROM) dir = (uint32_t)level >= o.bu_from;
        if (o.direction == IBFS_DIR_SCHEDULE && (uint32_t)level - 1 < o.schedule_len)
          dir = (o.schedule[level - 1] == 'B' || o.schedule[level - 1] == 1);
        scan((int)dir);
      }
      const uint32_t njfq = (uint32_t)h_ctr[0];
      CK(cudaMemsetAsync(newcnt, 0, W * 4, stream));
      if (njfq) {
        joint_expand<<<grid, 256, 0, stream>>>(a, level, (int)dir, njfq);
        launches++;
      }
      CK(cudaMemcpyAsync(h_new.data(), newcnt, W * 4, cudaMemcpyDeviceToHost, stream));
      CK(cudaMemcpyAsync(h_ctr, ctr, 32, cudaMemcpyDeviceToHost, stream));
      CK(cudaStreamSynchronize(stream));
      uint64_t np = 0;
      uint32_t nact[4] = {0, 0, 0, 0};
      for (uint32_t j = 0; j < W; ++j)
        if (h_new[j]) { np += h_new[j]; nact[j >> 5] |= 1u << (j & 31); }
      ibfs_level_stats &P = per_level[level - 1];
      if (dir) { P.bu_groups++; P.jfq_bu += njfq; st.levels_bu++; } else { P.td_groups++; P.jfq_td += njfq; st.levels_td++; }
      P.inspected += h_ctr[2];
      P.new_pairs += np;
      st.edges_inspected += h_ctr[2];
      st.max_levels = std::max<uint32_t>(st.max_levels, (uint32_t)level);
      if (level >= 128 && np) range_error = true;
      std::memcpy(act, nact, sizeof(act));
      if (o.max_depth && (uint32_t)level >= o.max_depth) break;  // k-hop (§8.7)
    }
    // rows (vertex-major JSA -> instance-major int8), isolated sources, m_s
    jsa_to_rows<<<grid, 256, 0, stream>>>(a, g->d_tbase, g->d_nzbits, nv, (int)rows, out);
    launches++;
    for (uint32_t j = 0; j < rows; ++j)
      if (csources[(size_t)gi * W + j] == NO_VERTEX)
        CK(cudaMemsetAsync(out + (size_t)j * nv + sources[(size_t)gi * W + j], 0, 1, stream));
    CK(cudaMemsetAsync(d_m, 0, W * 8, stream));
    jsa_ms<<<grid, W, 0, stream>>>(a, d_m);
    launches++;
    CK(cudaEventRecord(w1, stream));
    win.push_back({w0, w1});
    if (stats && stats->per_source_digest) {
      BatchArgs<uint32_t> b{};
      b.out = out;
      b.nv = nv;
      b.n_total = rows;
      b.group0 = 0;
      CK(cudaMemsetAsync(d_dig, 0, W * 8, stream));
      digest_kernel<uint32_t><<<dim3(64, rows), BLOCK, 0, stream>>>(b, d_dig);
      launches++;
      CK(cudaMemcpyAsync(h_dig.data(), d_dig, W * 8, cudaMemcpyDeviceToHost, stream));
    }
    CK(cudaMemcpyAsync(h_m.data(), d_m, W * 8, cudaMemcpyDeviceToHost, stream));
    if (out_host)
      CK(cudaMemcpyAsync(out_depths + (size_t)gi * W * nv, staging, (size_t)rows * nv, cudaMemcpyDeviceToHost, stream));
    CK(cudaStreamSynchronize(stream));
    for (uint32_t r = 0; r < rows; ++r) {
      st.edges_traversed += h_m[r];
      if (stats && stats->per_source_m) stats->per_source_m[(size_t)gi * W + r] = h_m[r];
      if (stats && stats->per_source_digest) stats->per_source_digest[(size_t)gi * W + r] = h_dig[r];
    }
  }
  if (range_error) fail(IBFS_E_RANGE, "a depth exceeds 127 (int8 output)");
  for (auto &p : win) { float ms = 0; CK(cudaEventElapsedTime(&ms, p.first, p.second)); st.traverse_ms += ms; }
  st.n_groups = n_groups;
  st.n_launches = launches;
  if (stats) {
    st.per_source_m = stats->per_source_m;
    st.per_source_digest = stats->per_source_digest;
    st.level_cap = stats->level_cap;
    st.per_level = stats->per_level;
    if (st.per_level)
      for (uint32_t i = 0; i < st.level_cap; ++i) st.per_level[i] = i < (uint32_t)MAXL ? per_level[i] : ibfs_level_stats{};
    *stats = st;
  }
}

}  // namespace

extern "C" int ibfs_run_ex(const ibfs_graph *g, const uint32_t *sources, uint32_t n, uint32_t group_bits,
                           int8_t *out_depths, const ibfs_run_opts *opts, ibfs_stats *stats) {
  const auto t_entry = HostClock::now();
  return guarded([&] {
    if (!g) fail(IBFS_E_INVALID, "graph is NULL");
    if (group_bits != 32 && group_bits != 64 && group_bits != 128) fail(IBFS_E_INVALID, "group_bits must be 32, 64 or 128");
    if (n > 0 && !sources) fail(IBFS_E_INVALID, "sources is NULL");
    ibfs_run_opts o;
    if (opts) o = *opts; else ibfs_run_opts_default(&o);
    if (o.direction > 3) fail(IBFS_E_INVALID, "bad direction mode");
    if (o.direction == IBFS_DIR_SCHEDULE && o.schedule_len > 0 && !o.schedule) fail(IBFS_E_INVALID, "schedule is NULL");
    if (!(o.alpha > 0) || !(o.beta > 0)) fail(IBFS_E_INVALID, "alpha and beta must be > 0");
    if (o.split > IBFS_SPLIT_FORCE) fail(IBFS_E_INVALID, "bad split mode");
    if (o.engine > IBFS_ENGINE_JOINT) fail(IBFS_E_INVALID, "bad engine");
    if (o.split == IBFS_SPLIT_FORCE && o.split_mod == 0) fail(IBFS_E_INVALID, "split_mod must be > 0");
    if (o.split == IBFS_SPLIT_AUTO && !(o.split_div > 0)) fail(IBFS_E_INVALID, "split_div must be > 0");
    if (stats) {
      if (stats->per_source_m) std::memset(stats->per_source_m, 0, (size_t)n * 8);
      if (stats->per_source_digest) std::memset(stats->per_source_digest, 0, (size_t)n * 8);
    }
    if (n == 0) {
      if (stats) {
        ibfs_stats z{};
        z.per_source_m = stats->per_source_m;
        z.per_source_digest = stats->per_source_digest;
        z.level_cap = stats->level_cap;
        z.per_level = stats->per_level;
        if (z.per_level) std::memset(z.per_level, 0, sizeof(ibfs_level_stats) * z.level_cap);
        *stats = z;
      }
      return;
    }
    DeviceScope ds(g->device);
    // sources: validate on the host.  Device-resident sources are read on the caller's
    // stream (ordered after the work that wrote them; torch streams are non-blocking
    // with respect to the legacy default stream)
    std::vector<uint32_t> hs(n), hcs(n);
    if (is_device_ptr(sources)) {
      CK(cudaMemcpyAsync(hs.data(), sources, (size_t)n * 4, cudaMemcpyDeviceToHost, (cudaStream_t)o.cuda_stream));
      CK(cudaStreamSynchronize((cudaStream_t)o.cuda_stream));
    } else {
      std::memcpy(hs.data(), sources, (size_t)n * 4);
    }
    for (uint32_t r = 0; r < n; ++r)
      if (hs[r] >= g->nv) fail(IBFS_E_INVALID, "source id >= nv");
    if (o.engine == IBFS_ENGINE_JOINT) {
      for (uint32_t r = 0; r < n; ++r) hcs[r] = host_compact_id(g, hs[r]);
      run_joint(g, hs.data(), hcs.data(), n, group_bits, out_depths, o, stats);
    } else if (group_bits == 32) run_typed<uint32_t>(g, hs.data(), n, out_depths, o, stats, t_entry);
    else if (group_bits == 64) run_typed<unsigned long long>(g, hs.data(), n, out_depths, o, stats, t_entry);
    else run_typed<u128>(g, hs.data(), n, out_depths, o, stats, t_entry);
  });
}

extern "C" int ibfs_run(const ibfs_graph *g, const uint32_t *sources, uint32_t n, uint32_t group_bits,
                        int8_t *out_depths) {
  return ibfs_run_ex(g, sources, n, group_bits, out_depths, nullptr, nullptr);
}
