/*
 * oracle/oracle.c -- TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load this library.  The
 * product path (paper_conf_sigmod_liuhh16_b200/) never imports, links or executes it,
 * and it shares no code, header, table or helper with the CUDA path.
 *
 * What it computes: the plain definition the paper's method reaches exactly
 * (PAPER.md P:L43-L49 shortest paths on unweighted graphs, Fig. 1
 * P:L151 BFS depths):
 *
 *     depth[r][v] = number of edges on a shortest path from sources[r] to v,
 *                   0 at the source, -1 if no path exists.
 *
 * Algorithm: one textbook FIFO-queue BFS per source (BACKGROUND: the
 * frontier queue starts with the source; each level inspects the neighbours of the
 * frontiers and marks the unvisited ones with depth + 1).  Adjacency is built from the
 * RAW tuple list, not from the GPU path's CSR: for a tuple (u, v) append v to adj[u],
 * and (undirected) u to adj[v]; duplicates and self-loops are kept.
 *
 * Also per source:
 *   m_s    = sum over reached v of |adj[v]|    (TEPS numerator, P:L887 / P:L977)
 *   digest = sum over reached v of splitmix64((v << 8) | (depth + 1))  mod 2^64
 *   ecc    = max depth, reached = number of reached vertices.
 * A depth > 127 (does not fit the int8 output) returns ORACLE_E_RANGE.
 *
 * Pins (tests/test_oracle.py): Floyd-Warshall brute force, closed forms, the paper's
 * worked example (tests/golden/fig1_depths.txt), scipy.sparse.csgraph, the complete
 * invariant certificate, APSP symmetry.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

#define ORACLE_OK 0
#define ORACLE_E_INVALID -1
#define ORACLE_E_NOMEM -2
#define ORACLE_E_RANGE -4

typedef struct {
  uint64_t nv;
  uint64_t *off;  /* [nv + 1] */
  uint32_t *adj;  /* [off[nv]] */
} oracle_graph;

void oracle_graph_free(oracle_graph *g) {
  if (!g) return;
  free(g->off);
  free(g->adj);
  free(g);
}

/* Build adjacency lists from the raw tuples, keeping tuple order within each list.
 * Thread t owns the vertex range [lo_t, hi_t) and scans every tuple twice (count, then
 * fill), appending only to its own lists -- the same sequential append order as a
 * single pass, just split by owner. */
typedef struct {
  uint64_t lo, hi, m;
  const uint32_t *u, *v;
  int directed, pass;
  uint64_t *off;   /* pass 0: counts at off[x + 1]; pass 1: fill cursors */
  uint32_t *adj;
} build_job;

static void *build_worker(void *arg) {
  build_job *j = (build_job *)arg;
  const uint64_t lo = j->lo, hi = j->hi;
  for (uint64_t e = 0; e < j->m; ++e) {
    uint32_t a = j->u[e], b = j->v[e];
    if (a >= lo && a < hi) {
      if (j->pass == 0) j->off[a + 1]++;
      else j->adj[j->off[a]++] = b;
    }
    if (!j->directed && b >= lo && b < hi) {
      if (j->pass == 0) j->off[b + 1]++;
      else j->adj[j->off[b]++] = a;
    }
  }
  return NULL;
}

oracle_graph *oracle_graph_new(uint64_t nv, uint64_t m, const uint32_t *u, const uint32_t *v,
                               int directed, int threads) {
  oracle_graph *g = (oracle_graph *)calloc(1, sizeof(oracle_graph));
  if (!g) return NULL;
  g->nv = nv;
  for (uint64_t e = 0; e < m; ++e)
    if (u[e] >= nv || v[e] >= nv) { free(g); return NULL; }
  g->off = (uint64_t *)calloc(nv + 1, sizeof(uint64_t));
  uint64_t entries = directed ? m : 2 * m;
  g->adj = (uint32_t *)malloc((entries ? entries : 1) * sizeof(uint32_t));
  uint64_t *cur = (uint64_t *)malloc((nv + 1) * sizeof(uint64_t));
  if (!g->off || !g->adj || !cur) { free(cur); oracle_graph_free(g); return NULL; }
  if (threads < 1) threads = 1;
  if (threads > 256) threads = 256;
  if ((uint64_t)threads > nv) threads = (int)nv;
  pthread_t tid[256];
  build_job jobs[256];
  for (int pass = 0; pass < 2; ++pass) {
    if (pass == 1) {
      for (uint64_t x = 0; x < nv; ++x) g->off[x + 1] += g->off[x];
      memcpy(cur, g->off, (nv + 1) * sizeof(uint64_t));
    }
    for (int t = 0; t < threads; ++t) {
      jobs[t].lo = nv * (uint64_t)t / (uint64_t)threads;
      jobs[t].hi = nv * (uint64_t)(t + 1) / (uint64_t)threads;
      jobs[t].m = m; jobs[t].u = u; jobs[t].v = v;
      jobs[t].directed = directed; jobs[t].pass = pass;
      jobs[t].off = pass == 0 ? g->off : cur;
      jobs[t].adj = g->adj;
    }
    for (int t = 1; t < threads; ++t) pthread_create(&tid[t], NULL, build_worker, &jobs[t]);
    build_worker(&jobs[0]);
    for (int t = 1; t < threads; ++t) pthread_join(tid[t], NULL);
  }
  free(cur);
  return g;
}

uint64_t oracle_graph_nv(const oracle_graph *g) { return g->nv; }
uint64_t oracle_graph_ne(const oracle_graph *g) { return g->off[g->nv]; }
/* Copy the adjacency out (for the numpy planner oracle and for tests). */
void oracle_graph_export(const oracle_graph *g, uint64_t *off, uint32_t *adj) {
  memcpy(off, g->off, (g->nv + 1) * sizeof(uint64_t));
  memcpy(adj, g->adj, g->off[g->nv] * sizeof(uint32_t));
}

static inline uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

typedef struct {
  const oracle_graph *g;
  const uint32_t *sources;
  uint64_t n;
  int8_t *out;        /* [n][nv] or NULL */
  uint64_t *m_s;      /* [n] or NULL */
  uint64_t *digest;   /* [n] or NULL */
  int32_t *ecc;       /* [n] or NULL */
  uint64_t *reached;  /* [n] or NULL */
  uint64_t next;      /* dynamic ticket */
  pthread_mutex_t lock;
  int status;
  int32_t kmax;       /* -1 = unbounded */
} bfs_job;

/* One textbook BFS from s into dist (int32, -1 = unvisited).  Returns max depth.
 * kmax >= 0 caps the search at the first kmax levels (the k-hop reachability index of
 * §8.7: "computes the first k levels BFS"): a vertex at depth kmax is
 * recorded but not expanded, so every vertex farther than kmax hops stays -1. */
static int32_t bfs_one(const oracle_graph *g, uint32_t s, int32_t kmax, int32_t *dist, uint32_t *queue,
                       uint64_t *m_out, uint64_t *dig_out, uint64_t *reached_out) {
  uint64_t head = 0, tail = 0;
  for (uint64_t x = 0; x < g->nv; ++x) dist[x] = -1;
  dist[s] = 0;
  queue[tail++] = s;
  int32_t ecc = 0;
  uint64_t m = 0, dig = 0;
  while (head < tail) {
    uint32_t x = queue[head++];
    int32_t dx = dist[x];
    if (dx > ecc) ecc = dx;
    m += g->off[x + 1] - g->off[x];
    dig += splitmix64(((uint64_t)x << 8) | (uint64_t)(dx + 1));
    if (kmax >= 0 && dx >= kmax) continue;
    for (uint64_t k = g->off[x]; k < g->off[x + 1]; ++k) {
      uint32_t w = g->adj[k];
      if (dist[w] == -1) {
        dist[w] = dx + 1;
        queue[tail++] = w;
      }
    }
  }
  *m_out = m;
  *dig_out = dig;
  *reached_out = tail;
  return ecc;
}

static void *bfs_worker(void *arg) {
  bfs_job *j = (bfs_job *)arg;
  const oracle_graph *g = j->g;
  int32_t *dist = (int32_t *)malloc((g->nv ? g->nv : 1) * sizeof(int32_t));
  uint32_t *queue = (uint32_t *)malloc((g->nv ? g->nv : 1) * sizeof(uint32_t));
  if (!dist || !queue) {
    pthread_mutex_lock(&j->lock);
    j->status = ORACLE_E_NOMEM;
    pthread_mutex_unlock(&j->lock);
    free(dist); free(queue);
    return NULL;
  }
  for (;;) {
    pthread_mutex_lock(&j->lock);
    uint64_t r = j->next++;
    pthread_mutex_unlock(&j->lock);
    if (r >= j->n) break;
    uint64_t m, dig, reached;
    int32_t ecc = bfs_one(g, j->sources[r], j->kmax, dist, queue, &m, &dig, &reached);
    if (ecc > 127) {
      pthread_mutex_lock(&j->lock);
      j->status = ORACLE_E_RANGE;
      pthread_mutex_unlock(&j->lock);
    }
    if (j->out) {
      int8_t *row = j->out + r * g->nv;
      for (uint64_t x = 0; x < g->nv; ++x) row[x] = (int8_t)(dist[x] > 127 ? 127 : dist[x]);
    }
    if (j->m_s) j->m_s[r] = m;
    if (j->digest) j->digest[r] = dig;
    if (j->ecc) j->ecc[r] = ecc;
    if (j->reached) j->reached[r] = reached;
  }
  free(dist);
  free(queue);
  return NULL;
}

/* Run n textbook BFSes (one per source) on `threads` worker threads, each capped at
 * max_depth levels (max_depth < 0: unbounded). */
int oracle_bfs_k(const oracle_graph *g, const uint32_t *sources, uint64_t n, int32_t max_depth, int8_t *out,
                 uint64_t *m_s, uint64_t *digest, int32_t *ecc, uint64_t *reached, int threads) {
  if (!g || (n && !sources)) return ORACLE_E_INVALID;
  for (uint64_t r = 0; r < n; ++r)
    if (sources[r] >= g->nv) return ORACLE_E_INVALID;
  if (threads < 1) threads = 1;
  if (threads > 1024) threads = 1024;
  if ((uint64_t)threads > n) threads = (int)(n ? n : 1);
  bfs_job job;
  job.g = g; job.sources = sources; job.n = n; job.out = out; job.m_s = m_s;
  job.digest = digest; job.ecc = ecc; job.reached = reached; job.next = 0;
  job.status = ORACLE_OK;
  job.kmax = max_depth < 0 ? -1 : max_depth;
  pthread_mutex_init(&job.lock, NULL);
  pthread_t *tid = (pthread_t *)malloc(sizeof(pthread_t) * (size_t)threads);
  if (!tid) return ORACLE_E_NOMEM;
  for (int t = 1; t < threads; ++t) pthread_create(&tid[t], NULL, bfs_worker, &job);
  bfs_worker(&job);
  for (int t = 1; t < threads; ++t) pthread_join(tid[t], NULL);
  free(tid);
  pthread_mutex_destroy(&job.lock);
  return job.status;
}

int oracle_bfs(const oracle_graph *g, const uint32_t *sources, uint64_t n, int8_t *out,
               uint64_t *m_s, uint64_t *digest, int32_t *ecc, uint64_t *reached, int threads) {
  return oracle_bfs_k(g, sources, n, -1, out, m_s, digest, ecc, reached, threads);
}

/* The complete BFS-depth certificate (the same four conditions as
 * oracle/certify.py, written as plain loops over the oracle's own adjacency so it checks
 * rows at config-5 scale).  Undirected graphs only.  Returns 0 if d is the exact BFS depth
 * row from s, else the number of the first violated condition:
 *   1 (o)   some d(v) < -1
 *   2 (i)   d(s) != 0
 *   3 (ii)  reachability differs across an edge
 *   4 (ii)  |d(u) - d(v)| > 1 across an edge
 *   5 (iii) a vertex other than s has depth 0
 *   6 (iii) a reached vertex v != s has no neighbour at d(v) - 1 */
int oracle_certify(const oracle_graph *g, uint32_t s, const int8_t *d) {
  const uint64_t nv = g->nv;
  if (s >= nv) return ORACLE_E_INVALID;
  for (uint64_t v = 0; v < nv; ++v)
    if (d[v] < -1) return 1;
  if (d[s] != 0) return 2;
  for (uint64_t u = 0; u < nv; ++u) {
    const int du = d[u];
    int has_pred = 0;
    for (uint64_t k = g->off[u]; k < g->off[u + 1]; ++k) {
      const int dv = d[g->adj[k]];
      if ((du == -1) != (dv == -1)) return 3;
      if (du >= 0 && (du - dv > 1 || dv - du > 1)) return 4;
      if (du >= 1 && dv == du - 1) has_pred = 1;
    }
    if (du == 0 && u != s) return 5;
    if (du >= 1 && !has_pred) return 6;
  }
  return 0;
}
