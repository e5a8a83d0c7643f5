/*
 * tdfs_inputs/gen.c -- seeded synthetic graph samplers shared by the oracle
 * tests and the CUDA path's tests/bench.
 *
 * This file holds NO arithmetic of the matching method (no intersection, no
 * backtracking, no CSR, no planner).  It only draws random edge lists and turns
 * them into a simple undirected graph (canonical (min,max) pairs, self-loops
 * dropped, duplicates removed, sorted).  Every random number is a pure function
 * of (seed, sample index) through splitmix64, so a run is bit-reproducible for
 * any thread count.
 *
 * Shapes follow SURVEY.md Appendix A.2 (R-MAT Graph500-style, Chung-Lu with a
 * power-law weight sequence) -- the synthetic stand-ins for the paper's Table I
 * datasets (Section IV-A).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>
#include <pthread.h>

static inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

/* Counter-based splitmix64 stream: the j-th draw of sample i under `seed`. */
static inline uint64_t draw(uint64_t seed, uint64_t i, uint64_t j) {
  uint64_t s = mix64(seed * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull);
  s = mix64(s ^ (i * 0xD1B54A32D192ED03ull));
  return mix64(s + (j + 1) * 0x9E3779B97F4A7C15ull);
}

static inline double unif(uint64_t x) { /* [0,1) with 53 bits */
  return (double)(x >> 11) * (1.0 / 9007199254740992.0);
}

/* ---------------------------------------------------------------- threads */
typedef struct {
  void (*fn)(void*, int64_t, int64_t);
  void* arg;
  int64_t lo, hi;
} job_t;

static void* job_run(void* p) {
  job_t* j = (job_t*)p;
  j->fn(j->arg, j->lo, j->hi);
  return NULL;
}

static void parallel_for(int64_t n, int nthreads, void (*fn)(void*, int64_t, int64_t), void* arg) {
  if (nthreads < 1) nthreads = 1;
  if (nthreads > 256) nthreads = 256;
  if (n < 65536 || nthreads == 1) { fn(arg, 0, n); return; }
  pthread_t th[256];
  job_t jobs[256];
  int64_t step = (n + nthreads - 1) / nthreads;
  int used = 0;
  for (int t = 0; t < nthreads; t++) {
    int64_t lo = t * step, hi = lo + step;
    if (lo >= n) break;
    if (hi > n) hi = n;
    jobs[t].fn = fn; jobs[t].arg = arg; jobs[t].lo = lo; jobs[t].hi = hi;
    pthread_create(&th[t], NULL, job_run, &jobs[t]);
    used++;
  }
  for (int t = 0; t < used; t++) pthread_join(th[t], NULL);
}

/* ------------------------------------------------------------------ R-MAT */
typedef struct {
  int scale; double a, b, c; uint64_t seed; uint64_t* keys; const int32_t* perm;
} rmat_arg;

static void rmat_body(void* p, int64_t lo, int64_t hi) {
  rmat_arg* r = (rmat_arg*)p;
  for (int64_t i = lo; i < hi; i++) {
    uint64_t u = 0, v = 0;
    for (int bit = 0; bit < r->scale; bit++) {
      double x = unif(draw(r->seed, (uint64_t)i, (uint64_t)bit));
      /* quadrant a: (0,0); b: (0,1); c: (1,0); d: (1,1) */
      uint64_t ub = (x >= r->a + r->b) ? 1u : 0u;
      uint64_t vb = ((x >= r->a && x < r->a + r->b) || x >= r->a + r->b + r->c) ? 1u : 0u;
      u |= ub << bit;
      v |= vb << bit;
    }
    uint64_t pu = (uint64_t)(uint32_t)r->perm[u], pv = (uint64_t)(uint32_t)r->perm[v];
    if (pu == pv) { r->keys[i] = UINT64_MAX; continue; }
    uint64_t lo_ = pu < pv ? pu : pv, hi_ = pu < pv ? pv : pu;
    r->keys[i] = (lo_ << 32) | hi_;
  }
}

/* -------------------------------------------------------------- Chung-Lu */
typedef struct {
  int64_t n; const double* cdf; uint64_t seed; uint64_t* keys; const int32_t* perm;
} cl_arg;

static inline int64_t cdf_pick(const double* cdf, int64_t n, double x) {
  /* smallest i with cdf[i] > x, cdf[n-1] == 1 */
  int64_t lo = 0, hi = n - 1;
  while (lo < hi) {
    int64_t mid = (lo + hi) >> 1;
    if (cdf[mid] > x) hi = mid; else lo = mid + 1;
  }
  return lo;
}

static void cl_body(void* p, int64_t lo, int64_t hi) {
  cl_arg* r = (cl_arg*)p;
  for (int64_t i = lo; i < hi; i++) {
    int64_t a = cdf_pick(r->cdf, r->n, unif(draw(r->seed, (uint64_t)i, 0)));
    int64_t b = cdf_pick(r->cdf, r->n, unif(draw(r->seed, (uint64_t)i, 1)));
    uint64_t pu = (uint64_t)(uint32_t)r->perm[a], pv = (uint64_t)(uint32_t)r->perm[b];
    if (pu == pv) { r->keys[i] = UINT64_MAX; continue; }
    uint64_t lo_ = pu < pv ? pu : pv, hi_ = pu < pv ? pv : pu;
    r->keys[i] = (lo_ << 32) | hi_;
  }
}

/* ------------------------------------------------- sort + dedupe of keys */
static void radix_sort_u64(uint64_t* a, int64_t n, int key_bits) {
  uint64_t* tmp = (uint64_t*)malloc((size_t)n * sizeof(uint64_t));
  if (!tmp) return;
  uint64_t* src = a; uint64_t* dst = tmp;
  int64_t* cnt = (int64_t*)malloc(sizeof(int64_t) * 65536);
  for (int shift = 0; shift < key_bits; shift += 16) {
    memset(cnt, 0, sizeof(int64_t) * 65536);
    for (int64_t i = 0; i < n; i++) cnt[(src[i] >> shift) & 0xFFFF]++;
    int64_t s = 0;
    for (int d = 0; d < 65536; d++) { int64_t c = cnt[d]; cnt[d] = s; s += c; }
    for (int64_t i = 0; i < n; i++) dst[cnt[(src[i] >> shift) & 0xFFFF]++] = src[i];
    uint64_t* t = src; src = dst; dst = t;
  }
  if (src != a) memcpy(a, src, (size_t)n * sizeof(uint64_t));
  free(cnt);
  free(tmp);
}

/* Sort keys, drop UINT64_MAX (self-loops) and duplicates; returns new length. */
static int64_t finish_keys(uint64_t* keys, int64_t n) {
  /* keys are (lo<<32)|hi with ids < 2^31, so 64 bits; UINT64_MAX sorts last */
  radix_sort_u64(keys, n, 64);
  int64_t w = 0;
  for (int64_t i = 0; i < n; i++) {
    if (keys[i] == UINT64_MAX) break;
    if (w > 0 && keys[w - 1] == keys[i]) continue;
    keys[w++] = keys[i];
  }
  return w;
}

static void perm_ids(int32_t* perm, int64_t n, uint64_t seed) {
  for (int64_t i = 0; i < n; i++) perm[i] = (int32_t)i;
  for (int64_t i = n - 1; i > 0; i--) { /* Fisher-Yates with counter draws */
    int64_t j = (int64_t)(draw(seed ^ 0xA5A5A5A5ull, (uint64_t)i, 7) % (uint64_t)(i + 1));
    int32_t t = perm[i]; perm[i] = perm[j]; perm[j] = t;
  }
}

/*
 * R-MAT: `nsamples` directed samples over 2^scale ids, ids randomly permuted
 * (so id order is uncorrelated with degree), canonicalised and deduplicated.
 * Writes up to nsamples keys ((u<<32)|v, u<v) into out_keys; returns count.
 */
int64_t tdfs_gen_rmat(int scale, int64_t nsamples, double a, double b, double c,
                      uint64_t seed, int nthreads, uint64_t* out_keys) {
  int64_t n = (int64_t)1 << scale;
  int32_t* perm = (int32_t*)malloc((size_t)n * sizeof(int32_t));
  if (!perm) return -1;
  perm_ids(perm, n, seed);
  rmat_arg r = {scale, a, b, c, seed, out_keys, perm};
  parallel_for(nsamples, nthreads, rmat_body, &r);
  free(perm);
  return finish_keys(out_keys, nsamples);
}

/*
 * Chung-Lu: weights w_i = wmax * ((i + i0) / i0)^(-1/(gamma-1)); endpoints drawn
 * i.i.d. proportional to w; ids permuted; canonicalised and deduplicated.
 */
int64_t tdfs_gen_chung_lu(int64_t n, int64_t nsamples, double gamma, double wmax, double i0,
                          uint64_t seed, int nthreads, uint64_t* out_keys) {
  double* cdf = (double*)malloc((size_t)n * sizeof(double));
  int32_t* perm = (int32_t*)malloc((size_t)n * sizeof(int32_t));
  if (!cdf || !perm) { free(cdf); free(perm); return -1; }
  double s = 0.0, ex = -1.0 / (gamma - 1.0);
  for (int64_t i = 0; i < n; i++) { s += wmax * pow(((double)i + i0) / i0, ex); cdf[i] = s; }
  for (int64_t i = 0; i < n; i++) cdf[i] /= s;
  cdf[n - 1] = 1.0;
  perm_ids(perm, n, seed);
  cl_arg r = {n, cdf, seed, out_keys, perm};
  parallel_for(nsamples, nthreads, cl_body, &r);
  free(cdf); free(perm);
  return finish_keys(out_keys, nsamples);
}

/* Sum of Chung-Lu weights for a given i0 (used to solve i0 so that sum = 2m). */
double tdfs_chung_lu_weight_sum(int64_t n, double gamma, double wmax, double i0) {
  double s = 0.0, ex = -1.0 / (gamma - 1.0);
  for (int64_t i = 0; i < n; i++) s += wmax * pow(((double)i + i0) / i0, ex);
  return s;
}

/* Generic canonicalise + dedupe of caller-provided keys (returns new length). */
int64_t tdfs_gen_finish(uint64_t* keys, int64_t n) { return finish_keys(keys, n); }

/* Uniform labels in [0, L): label of vertex i is a pure function of (seed, i). */
void tdfs_gen_labels(int64_t n, int L, uint64_t seed, uint8_t* out) {
  for (int64_t i = 0; i < n; i++) out[i] = (uint8_t)(draw(seed ^ 0x1AB31ull, (uint64_t)i, 3) % (uint64_t)L);
}
