/*
 * include/ibfs.h -- C ABI of libibfs.so: the joint bitwise traversal of i concurrent BFS
 * instances over one shared CSR graph (iBFS, Liu, Huang, Hu, SIGMOD'16 -- PAPER.md),
 * hand-written for B200 (sm_100a).
 *
 * Citations are PAPER.md lines of the page-by-page extraction ("P:L<n>") plus the section,
 * algorithm or equation they fall in.
 *
 * General conventions
 *  - Every entry point returns int: IBFS_OK (0) or a negative ibfs_status.  Nothing throws
 *    or exits across the ABI; ibfs_last_error() returns a thread-local message for the
 *    last failing call on the calling thread.
 *  - Validation happens before any device work; on error, output contents are unspecified.
 *  - Pointer arguments documented "host or device" are classified with
 *    cudaPointerGetAttributes (device / managed memory = device, anything else = host).
 *  - A loaded graph is read-only; concurrent ibfs_run* calls on one graph are allowed on
 *    distinct streams (each call owns its scratch memory).
 *  - There is no CPU fallback: with no usable CUDA device every compute entry point
 *    returns IBFS_E_CUDA.
 */
#ifndef IBFS_H
#define IBFS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  IBFS_OK = 0,
  IBFS_E_INVALID = -1,     /* bad argument (NULL, id >= nv, bad group_bits, bad CSR) */
  IBFS_E_NOMEM = -2,       /* device or host allocation failed */
  IBFS_E_CUDA = -3,        /* CUDA runtime error, or no usable device */
  IBFS_E_RANGE = -4,       /* some depth > 127 does not fit the int8 output */
  IBFS_E_UNSUPPORTED = -5  /* valid request this build does not implement (degree >= 2^32) */
} ibfs_status;

typedef struct ibfs_graph ibfs_graph; /* opaque; owned by the library */

/* Library version (major * 10000 + minor * 100 + patch). */
int ibfs_version(void);

/* Thread-local message describing the last failing call on this thread ("" if none). */
const char *ibfs_last_error(void);

/* ---------------------------------------------------------------- graph loading ----
 * Graph storage follows P:L977 (§8.1): CSR; "each edge is considered as two directed
 * edges" for undirected graphs; the edge sequence is preserved.
 *
 * ibfs_load_csr: copy a CSR into device memory owned by the library on `device`.
 *   offsets[nv + 1] (u64): offsets[0] = 0, non-decreasing, offsets[nv] = ne.
 *   adj[ne] (u32): every id < nv.  Undirected graphs pass the symmetrized CSR and
 *   rev_offsets = rev_adj = NULL (bottom-up reads the same rows).  Directed graphs pass
 *   the out-edge CSR in offsets/adj (top-down expands it) and its transpose, the in-edge
 *   CSR, in rev_offsets[nv + 1] / rev_adj[ne] ("for directed graphs, we also store the
 *   reverse edges"; bottom-up reads a vertex's parents from it).  The transpose
 *   is checked by degree sequences (every vertex's occurrences in adj == its rev row
 *   length and vice versa) -> IBFS_E_INVALID; it is not otherwise verified.
 *   Inputs may be host or device pointers; they are neither retained nor modified.
 *   nv >= 1, ne < 2^40.  On success *out_graph owns all device state; release with
 *   ibfs_free.
 */
int ibfs_load_csr(int device, uint32_t nv, uint64_t ne, const uint64_t *offsets,
                  const uint32_t *adj, const uint64_t *rev_offsets, const uint32_t *rev_adj,
                  ibfs_graph **out_graph);

/* ibfs_load_edges: build the CSR on the device from a tuple list (u[e], v[e]),
 *   e < n_tuples (host or device pointers).  Undirected (directed = 0): tuple (u, v)
 *   yields entries u->v and v->u; duplicates and self-loops are kept (a self-loop tuple
 *   gives two entries), and each row keeps tuple order (stable) -- P:L887.
 *   Directed (directed != 0): tuple (u, v) is the edge u->v only; the library builds
 *   the out-edge rows (top-down) and the in-edge rows (bottom-up), both in tuple order. */
int ibfs_load_edges(int device, uint32_t nv, uint64_t n_tuples, const uint32_t *u,
                    const uint32_t *v, int directed, ibfs_graph **out_graph);

/* Row order of the device adjacency (never changes any result).  Applies
 * to the rows bottom-up scans: the CSR of an undirected graph, the in-edge rows of a
 * directed one (keyed by the parent's in-degree).
 *   IBFS_ROWS_KEEP      keep the loaded order (tuple order for ibfs_load_edges).
 *   IBFS_ROWS_HUB_FIRST stable-sort every row by neighbour outdegree, descending, so
 *                       bottom-up inspection (Alg. 1) meets the vertices most
 *                       likely visited first and terminates early on hot words. */
enum { IBFS_ROWS_KEEP = 0, IBFS_ROWS_HUB_FIRST = 1 };
int ibfs_graph_sort_rows(ibfs_graph *g, int order);

/* Graph facts.  Any output pointer may be NULL. */
int ibfs_graph_info(const ibfs_graph *g, uint32_t *nv, uint64_t *ne, uint32_t *max_degree,
                    int *device);

/* Copy the device CSR (the out-edge rows of a directed graph) back to caller-allocated
 * HOST arrays offsets[nv+1], adj[ne]. */
int ibfs_graph_export_csr(const ibfs_graph *g, uint64_t *offsets, uint32_t *adj);

/* Release everything g owns.  NULL-safe. */
void ibfs_free(ibfs_graph *g);

/* ------------------------------------------------------------------- planning ----
 * Outdegree-based GroupBy, §5.2: Rule 1 "the out-degrees of these two
 * source vertices are less than p"; Rule 2 "two source vertices connect to at
 * least one common vertex whose outdegree is greater than q"; q = 128 and p
 * ascending over {4, 16, 64, 128} by default; full groups first, then combined
 * small groups, then the rest "in a random manner"; uniform graphs group by a
 * shared vertex of any degree.  The exact step order is DESIGN.md §2 reading #16.
 */
typedef struct {
  uint32_t mode;     /* 0 = GroupBy (default), 1 = seeded random, 2 = identity */
  uint32_t q;        /* hub: outdegree > q (default 128) */
  uint32_t n_p;      /* number of Rule-1 bounds in p[] (1..8; default 4) */
  uint32_t p[8];     /* ascending Rule-1 bounds (default 4, 16, 64, 128) */
  uint32_t hops;     /* 1 (default): the steps above.  2: "not required ... directly ... as long
                        as within the first several levels" -- the bucket leftovers and
                        the Rule-1 rejects that have a hub are ordered by their 2-hop anchor
                        (the larger of hub(r) and hub(hub(r)) by degree) before grouping */
  uint64_t seed;     /* seeded Fisher-Yates for the random remainder / random mode (3) */
} ibfs_plan_params;

void ibfs_plan_params_default(ibfs_plan_params *p);

/* out_perm[n] (caller-allocated host array) receives a permutation of 0..n-1, indices
 * into `sources` (host or device).  Group k = sources[out_perm[k*group_bits ..
 * k*group_bits + group_bits - 1]]; only the last group may be short.
 * *out_n_groups = ceil(n / group_bits).  group_bits in {32, 64, 128}.  params NULL =
 * defaults.  Runs a device kernel for the per-source hub search, the rest on the host.
 * Device-resident `sources` are read after a device-wide synchronize (every stream's
 * pending work, including the writer's, completes first). */
int ibfs_plan_groups(const ibfs_graph *g, const uint32_t *sources, uint32_t n,
                     uint32_t group_bits, const ibfs_plan_params *params, uint32_t *out_perm,
                     uint32_t *out_n_groups);

/* ------------------------------------------------------------------- traversal ----
 * ibfs_run: n BFS instances, one per entry of `sources` (host or device, each < nv;
 * duplicates allowed and give identical rows).  Each consecutive chunk of group_bits
 * sources is one group that shares one group_bits-wide status word per vertex -- the
 * Bitwise Status Array of §6 (Alg. 1, Alg. 2).
 * group_bits in {32, 64, 128} ("int, int4, long4" vector types P:L825-L829; N = 128
 * default).
 *
 * out_depths: int8 [n][nv] row-major, caller-allocated; row r holds the BFS depth of
 * every vertex from sources[r]: 0 at the source, -1 if unreachable (Fig. 1; our
 * depth = the paper's depth - 1, reading #1).  Host or device pointer, or
 * NULL (depths are still materialised in device scratch -- the timed window ends with
 * "the results ... stored in GPU memory", P:L887 -- and only statistics are returned).
 * n == 0 returns IBFS_OK and does nothing.  A depth > 127 returns IBFS_E_RANGE.
 * Runs on the legacy default stream and returns after the work completes.
 */
int ibfs_run(const ibfs_graph *g, const uint32_t *sources, uint32_t n, uint32_t group_bits,
             int8_t *out_depths);

enum {
  IBFS_DIR_AUTO = 0,      /* per-group switch from device counters (reading #7) */
  IBFS_DIR_TD_ONLY = 1,   /* top-down every level */
  IBFS_DIR_BU_FROM = 2,   /* top-down before level bu_from, bottom-up from it on */
  IBFS_DIR_SCHEDULE = 3   /* schedule[l-1] for level l ('T' or 'B'); auto beyond it */
};

typedef struct {
  uint32_t direction;         /* IBFS_DIR_* (default AUTO).  Never changes results. */
  uint32_t bu_from;           /* for IBFS_DIR_BU_FROM (level >= 1) */
  const uint8_t *schedule;    /* host array of 'T'/'B' for IBFS_DIR_SCHEDULE */
  uint32_t schedule_len;
  float alpha;                /* TD->BU when m_f * alpha > m_u (default 3.0) */
  float beta;                 /* BU->TD when n_f * beta < nv_active (default 24.0) */
  uint32_t groups_in_flight;  /* groups per launch batch; 0 = auto from nv and memory */
  void *cuda_stream;          /* cudaStream_t to launch on; NULL = legacy default stream.
                                 Device-resident sources are read on this stream, so work
                                 queued on it before the call (e.g. the kernel that wrote
                                 them) completes first. */
  uint32_t timing;            /* 1: CUDA events around every level kernel -> stats */
  /* Per-instance direction inside a bottom-up level (never changes results).  The paper
     runs one direction per group; a BU level stops early at a vertex only
     once every active instance's bit is found there, so one instance with a tiny
     frontier (a slow source, a small component) turns every row scan into a full one.
     IBFS_SPLIT_AUTO: in a BU level, the instances whose sampled frontier edge count m_f(j)
     satisfies m_f(j) * split_div < m_u(j) (their unexplored edges; Beamer's rule per
     instance) run top-down in the same launch. */
  uint32_t split;             /* IBFS_SPLIT_* (default AUTO) */
  uint32_t split_mod;         /* IBFS_SPLIT_FORCE: instances j with j % split_mod == 0 */
  float split_div;            /* IBFS_SPLIT_AUTO ratio (default 512) */
  /* k-hop mode (the reachability index of §8.7: "computes the first k
     levels BFS for a large amount of selected vertices"; Table 1 uses k = 3).  max_depth
     = k >= 1 stops every group after level k: vertices farther than k hops stay -1 and
     m_s counts the vertices within k hops.  0 = unbounded (plain BFS, the default). */
  uint32_t max_depth;
  /* Traversal engine.  IBFS_ENGINE_BITWISE (default): the bitwise status words of §6
      -- the product path.  IBFS_ENGINE_JOINT: the byte-per-instance Joint
     Status Array of §4 (one warp per vertex builds the JFQ, the lanes of a
     warp are the instances of a frontier), one group at a time with host-driven levels,
     kept as the "Joint" rung of the ablation ladder (Fig. 15).  Same results
     (max_depth included); split and groups_in_flight are bitwise-engine options. */
  uint32_t engine;
  /* Test hook: capacity of each group's late list -- the new vertices of sparse-committed
     levels, whose depths are written by a fix-up pass instead of the depth kernel reading
     their snapshot.  0 = default (non-isolated vertices / 32 + 1024).  A
     level whose entries do not fit is read from its snapshot instead; results never change. */
  uint32_t late_cap;
  uint32_t reserved;
} ibfs_run_opts;

enum { IBFS_ENGINE_BITWISE = 0, IBFS_ENGINE_JOINT = 1 };

enum {
  IBFS_SPLIT_AUTO = 0,   /* small-frontier instances of a BU level run top-down */
  IBFS_SPLIT_OFF = 1,    /* one direction per group per level, as in the paper */
  IBFS_SPLIT_FORCE = 2   /* tests: instances j % split_mod == 0 top-down in every BU level */
};

void ibfs_run_opts_default(ibfs_run_opts *o);

/* Per-level counters, summed over groups (our level l discovers depth l). */
typedef struct {
  uint32_t td_groups, bu_groups;  /* groups that ran this level top-down / bottom-up */
  uint64_t jfq_td, fq_td;         /* |JFQ| and sum_j |FQ_j| of the TD groups (Eq. 1) */
  uint64_t jfq_bu, fq_bu;         /* same for the BU groups (reading #23) */
  uint64_t inspected;             /* neighbour inspections (adjacency entries examined) */
  uint64_t new_pairs;             /* (instance, vertex) pairs discovered (depth == l) */
  uint64_t gathered;              /* neighbour status words actually read: bottom-up
                                     frontier-bitmap hits + top-down pre-checks */
  double expand_ms, commit_ms;    /* device time of this level's launches (opts.timing) */
} ibfs_level_stats;

typedef struct {
  double traverse_ms;          /* device time: group init + all level kernels */
  double finalize_ms;          /* m_s / digest pass (outside traverse_ms) */
  double copyout_ms;           /* device->host depth copies (host out_depths only) */
  uint64_t edges_traversed;    /* sum_s m_s: TEPS numerator (reading #11) */
  uint64_t edges_inspected;    /* neighbour inspections actually done (TD + BU) */
  uint64_t bytes_algorithmic;  /* DESIGN.md §5 byte model, all kernels */
  uint64_t sd_fq_td, sd_jfq_td, sd_fq_bu, sd_jfq_bu;  /* Eq. 1 numerators/denominators */
  uint32_t n_groups, max_levels;
  uint32_t levels_td, levels_bu;  /* group-levels run in each direction */
  uint64_t n_launches;            /* kernels this call launched (traversal + finalize) */
  /* per-kernel device time and algorithmic bytes.  One level_kernel launch per level runs
     the commit of level l-1 and the expand of level l (bytes: commit_bytes + expand_bytes);
     level_ms / init_ms / depth_ms are CUDA-event times (opts.timing only); expand_ms and
     commit_ms split level time by the kernel's own globaltimer stamps (always). */
  double level_ms, expand_ms, commit_ms, init_ms, depth_ms;
  uint64_t level_launches, init_launches, depth_launches;
  uint64_t expand_bytes, commit_bytes, init_bytes, depth_bytes;
  double level_gap_ms;  /* device idle between consecutive level kernels of a batch (in-kernel
                           globaltimer stamps): launch latency plus any host polling stall */
  /* Byte models (SURVEY.md §8(d) "Algorithmic bytes"):
     expand_bytes  per queued frontier 8 (row start) + B (its word); per inspection 4
                   (adjacency entry); per gathered neighbour word B (a bottom-up neighbour
                   is read only when the frontier bitmap holds it); per S_l write B; a
                   bottom-up level reads the frontier bitmap (nva/8) once;
     commit_bytes  the §8(d) dense-scan model: 2B per vertex and level (S_l and visited
                   read; 3B with IBFS_CLEAN_RING=0, where the commit also clears the next
                   slot) + B per vertex with new bits + the frontier bitmap written (nva/8);
     commit_bytes_moved  what the commits actually stream: a sparse commit
                   reads the chunk map, the marked chunks (bounded by the level's writes)
                   and clears the next slot;
     depth_bytes   depth_kernel only: int8 rows written (depth_rows_bytes) + B per vertex,
                   group and loaded snapshot level (levels 1..last_level of each group,
                   skipped levels excluded) + the late-list fix-ups; with the clean ring
                   at W = 128 the depth kernel also zeroes each loaded run (B per vertex,
                   group and loaded level, bulk stores) and clean_bytes excludes them;
     ms_bytes      the m_s pass: (B + 4) per vertex and group (final words + degrees); with
                   the clean ring also B per vertex and group (visited zeroed) and B per
                   vertex, group and loaded level of the final flush (the ring slots it
                   returns to zero; IBFS_MS_CLEAN=0 leaves them to ring_clean_kernel). */
  uint64_t commit_bytes_moved, depth_rows_bytes, ms_bytes;
  double ms_ms;                  /* m_s pass + late-list / isolated-source fix-ups (opts.timing) */
  uint64_t ms_launches;
  uint64_t level_launches_live;  /* level launches in which a group was still running (the
                                    others are look-ahead launches that exit at once) */
  uint64_t words_gathered;       /* sum of ibfs_level_stats.gathered */
  /* host-side wall clock of the call (diagnostics of the gaps between device work):
     entry -> the first kernel enqueued, time blocked waiting on the device, entry -> return */
  double host_setup_ms, host_wait_ms, host_total_ms;
  /* clean ring: ring_clean_kernel zeroes the snapshot slots the depth pass
     read (B per vertex, group and loaded level) and late_fix_kernel the skipped levels'
     entries (B each), so no commit clears a slot; clean_ms is CUDA-event time (opts.timing) */
  double clean_ms;
  uint64_t clean_launches, clean_bytes;
  /* optional caller-provided HOST arrays (NULL = not wanted) */
  uint64_t *per_source_m;       /* [n] m_s */
  uint64_t *per_source_digest;  /* [n] sum over reached v of splitmix64((v<<8)|(d+1)) */
  uint32_t level_cap;           /* capacity of per_level */
  ibfs_level_stats *per_level;  /* [level_cap]; entry l-1 = level l */
} ibfs_stats;

/* ibfs_run with options and statistics.  opts / stats may be NULL.  The caller owns
 * the arrays stats->per_source_* / per_level; the library zero-fills and writes them. */
int ibfs_run_ex(const ibfs_graph *g, const uint32_t *sources, uint32_t n, uint32_t group_bits,
                int8_t *out_depths, const ibfs_run_opts *opts, ibfs_stats *stats);

/* -------------------------------------------------------------------- memory ----
 * Route the library's device scratch through a caller allocator (Python installs
 * torch's caching allocator).  alloc(bytes, device, ctx) returns a device pointer or
 * NULL; release(ptr, device, ctx).  Pass alloc = release = NULL to restore the default
 * (stream-ordered cudaMallocAsync pool).  Process-wide; not for concurrent swapping. */
int ibfs_set_allocator(void *(*alloc)(size_t bytes, int device, void *ctx),
                       void (*release)(void *ptr, int device, void *ctx), void *ctx);

#ifdef __cplusplus
}
#endif
#endif /* IBFS_H */
