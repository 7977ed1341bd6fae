/*
 * ibfs_gen/gen.c -- seeded synthetic INPUT generator shared by the oracle and the
 * CUDA path (the only code both sides may use).  It holds none of the method's
 * arithmetic: it draws R-MAT / Kronecker edge tuples, a seeded vertex relabeling
 * and a seeded source sample, nothing else.
 *
 * Recipe (SURVEY.md §8(d) "Generator spec"):
 *   - tuple e in [0, M), M = ef * 2^scale; for each bit b in [0, scale) one 64-bit
 *     counter-based draw h = mix64(mix64(seed + GOLDEN) ^ ((e << 6) | b)) gives two
 *     32-bit uniforms r1 = hi32(h) / 2^32, r2 = lo32(h) / 2^32 (compared exactly as
 *     integers against floor(p * 2^32));
 *     ii = r1 > A+B, jj = r2 > (ii ? C/(C+D) : A/(A+B)); u |= ii << b, v |= jj << b.
 *     The quadrant probabilities are then A, B, C, D (PAPER.md P:L975 gives
 *     (A,B,C) = (0.57,0.19,0.19) for the Graph500 "KG" graphs and (0.45,0.15,0.15)
 *     for "RM").
 *   - relabeling: seeded Fisher-Yates permutation pi of [0, 2^scale) applied to both
 *     endpoints (draw j = mulhi64(mix64(k2 ^ i), i + 1)).
 *   - duplicates and self-loops are kept; tuples are not shuffled (P:L977 keeps the
 *     edge sequence).
 *   - sources: seeded Fisher-Yates over the ascending list of vertices that appear in
 *     at least one tuple (deg > 0); take the first i.
 * Every draw is a pure function of (seed, counter), so the output does not depend on
 * the thread count.
 */
#include <stdint.h>
#include <stddef.h>
#include <stdlib.h>
#include <string.h>
#include <pthread.h>

static inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

#define GOLDEN 0x9E3779B97F4A7C15ULL
#define PERM_SALT 0x5851F42D4C957F2DULL

static inline uint64_t mulhi64(uint64_t a, uint64_t b) {
  return (uint64_t)(((__uint128_t)a * (__uint128_t)b) >> 64);
}

typedef struct {
  uint64_t e0, e1;
  int scale;
  uint64_t key;
  uint64_t t_ab, t_c_cd, t_a_ab; /* floor(p * 2^32): r > p  <=>  (r * 2^32) > floor(p * 2^32) */
  uint32_t *u, *v;
  const uint32_t *perm;
} rmat_job;

static void *rmat_worker(void *arg) {
  rmat_job *j = (rmat_job *)arg;
  for (uint64_t e = j->e0; e < j->e1; ++e) {
    uint32_t u = 0, v = 0;
    for (int b = 0; b < j->scale; ++b) {
      uint64_t h = mix64(j->key ^ ((e << 6) | (uint64_t)b));
      uint64_t r1 = h >> 32, r2 = h & 0xffffffffULL;
      uint32_t ii = r1 > j->t_ab;
      uint32_t jj = r2 > (ii ? j->t_c_cd : j->t_a_ab);
      u |= ii << b;
      v |= jj << b;
    }
    if (j->perm) { u = j->perm[u]; v = j->perm[v]; }
    j->u[e] = u;
    j->v[e] = v;
  }
  return NULL;
}

/* floor(p * 2^32) as an integer threshold (exact: for integer r, r > x <=> r > floor(x)). */
static uint64_t thresh(double p) {
  double x = p * 4294967296.0;
  if (x >= 4294967296.0) return 4294967296ULL;
  if (x <= 0) return 0;
  return (uint64_t)x;
}

/* Fisher-Yates permutation of [0, n): out[i] = pi(i). */
void ibfs_gen_permutation(uint64_t n, uint64_t seed, uint32_t *out) {
  uint64_t k2 = mix64(seed ^ PERM_SALT);
  for (uint64_t i = 0; i < n; ++i) out[i] = (uint32_t)i;
  for (uint64_t i = n; i-- > 1;) {
    uint64_t j = mulhi64(mix64(k2 ^ i), i + 1);
    uint32_t t = out[i]; out[i] = out[j]; out[j] = t;
  }
}

/* R-MAT tuples, relabeled by the seeded permutation when relabel != 0.
 * u, v: caller-allocated [ef << scale].  Returns 0, or -1 on bad arguments. */
int ibfs_gen_rmat(int scale, uint32_t edgefactor, double A, double B, double C,
                  uint64_t seed, int relabel, int threads, uint32_t *u, uint32_t *v) {
  if (scale < 1 || scale > 31 || !u || !v || edgefactor == 0) return -1;
  double D = 1.0 - A - B - C;
  if (A < 0 || B < 0 || C < 0 || D < 0 || A + B <= 0 || C + D <= 0) return -1;
  uint64_t nv = 1ULL << scale;
  uint64_t m = (uint64_t)edgefactor << scale;
  uint32_t *perm = NULL;
  if (relabel) {
    perm = (uint32_t *)malloc(nv * sizeof(uint32_t));
    if (!perm) return -1;
    ibfs_gen_permutation(nv, seed, perm);
  }
  if (threads < 1) threads = 1;
  if (threads > 256) threads = 256;
  pthread_t tid[256];
  rmat_job jobs[256];
  uint64_t key = mix64(seed + GOLDEN);
  for (int t = 0; t < threads; ++t) {
    jobs[t].e0 = m * (uint64_t)t / (uint64_t)threads;
    jobs[t].e1 = m * (uint64_t)(t + 1) / (uint64_t)threads;
    jobs[t].scale = scale;
    jobs[t].key = key;
    jobs[t].t_ab = thresh(A + B);
    jobs[t].t_c_cd = thresh(C / (C + D));
    jobs[t].t_a_ab = thresh(A / (A + B));
    jobs[t].u = u;
    jobs[t].v = v;
    jobs[t].perm = perm;
  }
  for (int t = 1; t < threads; ++t) pthread_create(&tid[t], NULL, rmat_worker, &jobs[t]);
  rmat_worker(&jobs[0]);
  for (int t = 1; t < threads; ++t) pthread_join(tid[t], NULL);
  free(perm);
  return 0;
}

/* Sources: seeded Fisher-Yates over the ascending list of vertices touched by at
 * least one tuple; the first `count` entries go to out.  Returns the number written
 * (min(count, #touched)). */
uint64_t ibfs_gen_sources(uint64_t nv, uint64_t m, const uint32_t *u, const uint32_t *v,
                          uint64_t count, uint64_t seed, uint32_t *out) {
  uint8_t *touched = (uint8_t *)calloc(nv, 1);
  if (!touched) return 0;
  for (uint64_t e = 0; e < m; ++e) { touched[u[e]] = 1; touched[v[e]] = 1; }
  uint64_t k = 0;
  for (uint64_t x = 0; x < nv; ++x) k += touched[x];
  uint32_t *list = (uint32_t *)malloc((k ? k : 1) * sizeof(uint32_t));
  if (!list) { free(touched); return 0; }
  k = 0;
  for (uint64_t x = 0; x < nv; ++x) if (touched[x]) list[k++] = (uint32_t)x;
  free(touched);
  uint64_t k2 = mix64(seed ^ PERM_SALT);
  for (uint64_t i = k; i-- > 1;) {
    uint64_t j = mulhi64(mix64(k2 ^ i), i + 1);
    uint32_t t = list[i]; list[i] = list[j]; list[j] = t;
  }
  uint64_t w = count < k ? count : k;
  memcpy(out, list, w * sizeof(uint32_t));
  free(list);
  return w;
}
