/*
 * rmat.c -- deterministic R-MAT / Kronecker graph generator (seeded input
 * generator shared by the oracle and the CUDA path; it holds none of the
 * eIM method's arithmetic).
 *
 * Recipe:
 *   scale s = ceil(log2 n); each "attempt" t = 0, 1, 2, ... draws one edge
 *   (src, dst) in [0, 2^s)^2 by descending s levels of the 2x2 quadrant
 *   recursion with probabilities (a, b, c, d = 1-a-b-c)  [rows = src];
 *   both ends go through one seeded uniform permutation of [0, 2^s); the
 *   attempt is kept iff src < n, dst < n and src != dst.  The graph is the
 *   first m DISTINCT kept (src, dst) pairs in attempt order.  Output is the
 *   reverse CSR (in-neighbour lists, rows ascending): in_off[n+1] (u64),
 *   in_nbr[m] (u32, ascending within each row).
 * Every random number is a pure function of (seed, attempt, word), so the
 * result does not depend on the thread count.
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static inline uint64_t mix64(uint64_t z) {
  z += 0x9e3779b97f4a7c15ULL;
  z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
  z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
  return z ^ (z >> 31);
}

static inline uint64_t rnd(uint64_t seed_h, uint64_t t, uint64_t word) {
  return mix64(seed_h ^ mix64(t * 64u + word));
}

typedef struct {
  uint32_t n, s;
  uint64_t seed_h;
  uint32_t ta, tab, tabc;
  const uint32_t* perm;
  uint64_t t0, t1;
  uint64_t* keys;  /* (dst << 32) | src */
  uint64_t* idx;   /* attempt index */
  uint64_t cnt;
  int oom;
} gen_job;

static void* gen_worker(void* arg) {
  gen_job* j = (gen_job*)arg;
  /* kept attempts are held in buffers grown on demand (not sized by the
   * attempt count: at C4/C5 that would be ~3x the kept edges) */
  uint64_t cap = (j->t1 - j->t0) / 4 + 1024;
  j->keys = (uint64_t*)malloc(cap * sizeof(uint64_t));
  j->idx = (uint64_t*)malloc(cap * sizeof(uint64_t));
  j->cnt = 0;
  j->oom = 0;
  for (uint64_t t = j->t0; t < j->t1; ++t) {
    uint32_t src = 0, dst = 0;
    uint64_t r64 = 0;
    for (uint32_t lvl = 0; lvl < j->s; ++lvl) {
      if ((lvl & 1) == 0) r64 = rnd(j->seed_h, t, lvl >> 1);  /* one 64-bit word per two levels */
      uint32_t r = (lvl & 1) ? (uint32_t)(r64 >> 32) : (uint32_t)r64;
      /* quadrant: [0,ta) -> (0,0), [ta,tab) -> (0,1), [tab,tabc) -> (1,0), else (1,1) */
      const uint32_t ga = r >= j->ta, gb = r >= j->tab, gc = r >= j->tabc;
      const uint32_t sb = gb, db = ga ^ gb ^ gc;
      src = (src << 1) | sb;
      dst = (dst << 1) | db;
    }
    src = j->perm[src];
    dst = j->perm[dst];
    if (src >= j->n || dst >= j->n || src == dst) continue;
    if (j->cnt == cap) {
      cap += cap / 2;
      uint64_t* k2 = (uint64_t*)realloc(j->keys, cap * sizeof(uint64_t));
      if (k2) j->keys = k2;
      uint64_t* i2 = k2 ? (uint64_t*)realloc(j->idx, cap * sizeof(uint64_t)) : NULL;
      if (!i2) { j->oom = 1; return NULL; }
      j->idx = i2;
    }
    j->keys[j->cnt] = ((uint64_t)dst << 32) | src;
    j->idx[j->cnt] = t;
    j->cnt++;
  }
  return NULL;
}

/* stable LSD radix sort of (key, idx) by key over [0, N) (single thread);
 * k2/i2 are scratch of N entries; the result ends in keys/idx. */
static void lsd_sort(uint64_t* keys, uint64_t* idx, uint64_t* k2, uint64_t* i2, uint64_t N, int key_bits) {
  const int DB = 11;
  const uint64_t NB = 1u << DB;
  uint64_t cnt[1u << 11];
  uint64_t *ka = keys, *ia = idx, *kb = k2, *ib = i2;
  for (int shift = 0; shift < key_bits; shift += DB) {
    memset(cnt, 0, sizeof(cnt));
    for (uint64_t i = 0; i < N; ++i) cnt[(ka[i] >> shift) & (NB - 1)]++;
    uint64_t sum = 0;
    for (uint64_t b = 0; b < NB; ++b) { uint64_t c = cnt[b]; cnt[b] = sum; sum += c; }
    for (uint64_t i = 0; i < N; ++i) {
      uint64_t p = cnt[(ka[i] >> shift) & (NB - 1)]++;
      kb[p] = ka[i];
      ib[p] = ia[i];
    }
    uint64_t* t;
    t = ka; ka = kb; kb = t;
    t = ia; ia = ib; ib = t;
  }
  if (ka != keys) {
    memcpy(keys, ka, N * sizeof(uint64_t));
    memcpy(idx, ia, N * sizeof(uint64_t));
  }
}

/* Parallel stable sort of (key, idx) by key: a stable partition on the top
 * PB key bits (per-thread counts over contiguous chunks, chunk order kept),
 * then every bucket LSD-sorted on the remaining bits by a pool of threads.
 * Equal keys keep their input order, exactly as a sequential stable sort. */
typedef struct {
  uint64_t *keys, *idx, *k2, *i2;
  uint64_t N, lo, hi;
  int T, t, key_bits, low_bits, PB;
  uint64_t* cnt;              /* T x NBK */
  uint64_t* bstart;           /* NBK + 1 */
  volatile uint64_t* next_b;  /* bucket claim counter (phase 3) */
  pthread_mutex_t* mu;
  int phase;
} sort_job;

static void* sort_worker(void* arg) {
  sort_job* j = (sort_job*)arg;
  const uint64_t NBK = 1ull << j->PB;
  uint64_t* c = j->cnt + (uint64_t)j->t * NBK;
  if (j->phase == 1) {
    for (uint64_t i = j->lo; i < j->hi; ++i) c[j->keys[i] >> j->low_bits]++;
  } else if (j->phase == 2) {
    for (uint64_t i = j->lo; i < j->hi; ++i) {
      uint64_t p = c[j->keys[i] >> j->low_bits]++;
      j->k2[p] = j->keys[i];
      j->i2[p] = j->idx[i];
    }
  } else {
    for (;;) {
      pthread_mutex_lock(j->mu);
      uint64_t b = (*j->next_b)++;
      pthread_mutex_unlock(j->mu);
      if (b >= NBK) break;
      uint64_t a = j->bstart[b], e = j->bstart[b + 1];
      /* bucket data is in k2/i2; sort it there with keys/idx as scratch */
      if (e > a) lsd_sort(j->k2 + a, j->i2 + a, j->keys + a, j->idx + a, e - a, j->low_bits);
    }
  }
  return NULL;
}

static int radix_sort(uint64_t* keys, uint64_t* idx, uint64_t N, int key_bits, int T) {
  uint64_t* k2 = (uint64_t*)malloc((N ? N : 1) * sizeof(uint64_t));
  uint64_t* i2 = (uint64_t*)malloc((N ? N : 1) * sizeof(uint64_t));
  if (!k2 || !i2) { free(k2); free(i2); return -1; }
  if (T < 1) T = 1;
  const int PB = key_bits < 11 ? key_bits : 11;
  const uint64_t NBK = 1ull << PB;
  uint64_t* cnt = (uint64_t*)calloc((size_t)T * NBK, sizeof(uint64_t));
  uint64_t* bstart = (uint64_t*)calloc(NBK + 1, sizeof(uint64_t));
  sort_job* jobs = (sort_job*)calloc((size_t)T, sizeof(sort_job));
  pthread_t* th = (pthread_t*)calloc((size_t)T, sizeof(pthread_t));
  pthread_mutex_t mu = PTHREAD_MUTEX_INITIALIZER;
  volatile uint64_t next_b = 0;
  if (!cnt || !bstart || !jobs || !th) { free(k2); free(i2); free(cnt); free(bstart); free(jobs); free(th); return -1; }
  for (int phase = 1; phase <= 3; ++phase) {
    if (phase == 2) {  /* exclusive offsets: bucket-major, thread (= chunk) order within a bucket */
      uint64_t sum = 0;
      for (uint64_t b = 0; b < NBK; ++b) {
        bstart[b] = sum;
        for (int t = 0; t < T; ++t) { uint64_t c = cnt[(uint64_t)t * NBK + b]; cnt[(uint64_t)t * NBK + b] = sum; sum += c; }
      }
      bstart[NBK] = sum;
    }
    for (int t = 0; t < T; ++t) {
      sort_job* j = &jobs[t];
      j->keys = keys; j->idx = idx; j->k2 = k2; j->i2 = i2; j->N = N;
      j->lo = N * (uint64_t)t / (uint64_t)T;
      j->hi = N * (uint64_t)(t + 1) / (uint64_t)T;
      j->T = T; j->t = t; j->key_bits = key_bits; j->low_bits = key_bits - PB; j->PB = PB;
      j->cnt = cnt; j->bstart = bstart; j->next_b = &next_b; j->mu = &mu; j->phase = phase;
      pthread_create(&th[t], NULL, sort_worker, j);
    }
    for (int t = 0; t < T; ++t) pthread_join(th[t], NULL);
  }
  /* sorted data is in k2/i2 */
  memcpy(keys, k2, N * sizeof(uint64_t));
  memcpy(idx, i2, N * sizeof(uint64_t));
  free(k2); free(i2); free(cnt); free(bstart); free(jobs); free(th);
  return 0;
}

static int cmp_u64(const void* a, const void* b) {
  uint64_t x = *(const uint64_t*)a, y = *(const uint64_t*)b;
  return (x > y) - (x < y);
}

/* k-th smallest (0-based) of v[0..N) ; v is permuted */
static uint64_t select_kth(uint64_t* v, uint64_t N, uint64_t kk) {
  int64_t lo = 0, hi = (int64_t)N - 1, k = (int64_t)kk;
  uint64_t state = 0x1234567ULL;
  while (hi > lo) {
    if (hi - lo < 64) {
      qsort(v + lo, (size_t)(hi - lo + 1), sizeof(uint64_t), cmp_u64);
      return v[k];
    }
    state = mix64(state);
    uint64_t pivot = v[lo + (int64_t)(state % (uint64_t)(hi - lo + 1))];
    int64_t i = lo, lt = lo, gt = hi;
    while (i <= gt) {
      if (v[i] < pivot) { uint64_t t = v[i]; v[i] = v[lt]; v[lt] = t; i++; lt++; }
      else if (v[i] > pivot) { uint64_t t = v[i]; v[i] = v[gt]; v[gt] = t; gt--; }
      else i++;
    }
    if (k < lt) hi = lt - 1;
    else if (k > gt) lo = gt + 1;
    else return pivot;
  }
  return v[k];
}

/* Returns 0 on success, -1 on bad args / OOM. */
int rmat_generate(uint32_t n, uint64_t m, double a, double b, double c, uint64_t seed,
                  int nthreads, uint64_t* in_off, uint32_t* in_nbr) {
  if (n < 2 || a < 0 || b < 0 || c < 0 || a + b + c > 1.0) return -1;
  if (m > (uint64_t)n * (uint64_t)(n - 1)) return -1;
  if (nthreads < 1) nthreads = 1;
  uint32_t s = 0;
  while (((uint64_t)1 << s) < n) s++;
  uint64_t N2 = (uint64_t)1 << s;
  uint64_t seed_h = mix64(seed ^ 0x52c0ffee5eedULL);
  /* seeded Fisher-Yates permutation of [0, 2^s) */
  uint32_t* perm = (uint32_t*)malloc(N2 * sizeof(uint32_t));
  if (!perm) return -1;
  for (uint64_t i = 0; i < N2; ++i) perm[i] = (uint32_t)i;
  for (uint64_t i = N2 - 1; i > 0; --i) {
    uint64_t r = mix64(seed_h ^ mix64(0xfeedULL << 40 | i));
    uint64_t jj = (uint64_t)(((unsigned __int128)r * (i + 1)) >> 64);
    uint32_t t = perm[i]; perm[i] = perm[jj]; perm[jj] = t;
  }
  const double two32 = 4294967296.0;
  uint32_t ta = (uint32_t)fmin(floor(a * two32), 4294967295.0);
  uint32_t tab = (uint32_t)fmin(floor((a + b) * two32), 4294967295.0);
  uint32_t tabc = (uint32_t)fmin(floor((a + b + c) * two32), 4294967295.0);
  if (m == 0) {
    for (uint32_t v = 0; v <= n; ++v) in_off[v] = 0;
    free(perm);
    return 0;
  }
  double frac = (double)n / (double)N2;
  uint64_t attempts = (uint64_t)(1.15 * (double)m / (frac * frac)) + 1024;
  for (;;) {
    gen_job* jobs = (gen_job*)calloc((size_t)nthreads, sizeof(gen_job));
    pthread_t* th = (pthread_t*)calloc((size_t)nthreads, sizeof(pthread_t));
    for (int t = 0; t < nthreads; ++t) {
      gen_job* j = &jobs[t];
      j->n = n; j->s = s; j->seed_h = seed_h; j->ta = ta; j->tab = tab; j->tabc = tabc;
      j->perm = perm;
      j->t0 = attempts * (uint64_t)t / (uint64_t)nthreads;
      j->t1 = attempts * (uint64_t)(t + 1) / (uint64_t)nthreads;
      pthread_create(&th[t], NULL, gen_worker, j);
    }
    uint64_t total = 0;
    int oom = 0;
    for (int t = 0; t < nthreads; ++t) {
      pthread_join(th[t], NULL);
      total += jobs[t].cnt;
      oom |= jobs[t].oom || !jobs[t].keys || !jobs[t].idx;
    }
    uint64_t* keys = oom ? NULL : (uint64_t*)malloc((total ? total : 1) * sizeof(uint64_t));
    uint64_t* idx = oom ? NULL : (uint64_t*)malloc((total ? total : 1) * sizeof(uint64_t));
    if (!keys || !idx) {
      for (int t = 0; t < nthreads; ++t) { free(jobs[t].keys); free(jobs[t].idx); }
      free(keys); free(idx); free(jobs); free(th); free(perm);
      return -1;
    }
    uint64_t pos = 0;
    for (int t = 0; t < nthreads; ++t) {
      memcpy(keys + pos, jobs[t].keys, jobs[t].cnt * sizeof(uint64_t));
      memcpy(idx + pos, jobs[t].idx, jobs[t].cnt * sizeof(uint64_t));
      pos += jobs[t].cnt;
      free(jobs[t].keys); free(jobs[t].idx);
    }
    free(jobs); free(th);
    if (radix_sort(keys, idx, total, 32 + (int)s, nthreads) != 0) return -1;
    /* unique keys, keeping the first attempt (stable sort => smallest idx first) */
    uint64_t u = 0;
    for (uint64_t i = 0; i < total; ++i) {
      if (i > 0 && keys[i] == keys[i - 1]) continue;
      keys[u] = keys[i];
      idx[u] = idx[i];
      u++;
    }
    if (u < m) {
      free(keys); free(idx);
      attempts = attempts + attempts / 2;
      continue;
    }
    uint64_t cutoff = ~0ULL;
    if (u > m) {
      uint64_t* tmp = (uint64_t*)malloc(u * sizeof(uint64_t));
      memcpy(tmp, idx, u * sizeof(uint64_t));
      cutoff = select_kth(tmp, u, m - 1);
      free(tmp);
    }
    memset(in_off, 0, ((uint64_t)n + 1) * sizeof(uint64_t));
    uint64_t e = 0;
    for (uint64_t i = 0; i < u; ++i) {
      if (idx[i] > cutoff) continue;
      uint32_t dst = (uint32_t)(keys[i] >> 32);
      in_off[dst + 1]++;
      in_nbr[e++] = (uint32_t)keys[i];
    }
    for (uint32_t v = 0; v < n; ++v) in_off[v + 1] += in_off[v];
    free(keys); free(idx); free(perm);
    return e == m ? 0 : -1;
  }
}
