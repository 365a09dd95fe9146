/*
 * workload/gen.c — seeded, counter-based synthetic input generators.
 *
 * This module is SHARED INPUT PLUMBING: both the CPU oracle (oracle/) and the
 * CUDA path (paper_conf_eurosys_xiellwgrs22_b200/) consume what it produces.
 * It holds NONE of the method's arithmetic (no flat-key coding, no hashing into
 * cache sets, no hit/miss/eviction logic, no pooling): only
 *   - embedding-table VALUES   E_t[row][col]           (Table 2: fp32 rows)
 *   - power-law feature IDs    (t, position) -> row    ("power law distribution",
 *                                                        alpha = -1.2; BASELINE a = 1.05 / 0.8-1.2)
 *   - bag lengths for multi-hot sum-pooled inputs      (P:L256-258 pooling; BASELINE cfg4)
 * Every stream is a pure function of (seed, coordinates), so Python, C and any
 * other consumer regenerate identical inputs without storing them.
 *
 * Zipf sampling: bounded rank-Zipf P(r) ∝ r^-a, r in [1, n], drawn by
 * rejection-inversion (Hörmann & Derflinger 1996).
 * Hot ranks are scattered over rows by a keyed bijection on [0, 2^f) with
 * cycle-walking.
 */
#include <math.h>
#include <stdint.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define EXPORT __attribute__((visibility("default")))

/* ---- counter-based mixing ------------------------------------------------ */
static inline uint64_t sm64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
static inline double u01(uint64_t x) { return (double)(sm64(x) >> 11) * 0x1.0p-53; }

EXPORT uint64_t flg_splitmix64(uint64_t x) { return sm64(x); }
EXPORT double flg_u01(uint64_t x) { return u01(x); }

/* ---- values -------------------------------------------------------------- */
/* mode 0 = grid: multiples of 2^-12 in [-0.5, 0.5): every fp32 sum of <= 4096
 *          such values is exact in any order (pooling parity, SURVEY c-6).
 * mode 1 = bits: arbitrary fp32 bit patterns (keeps +-0, denormals; no Inf/NaN):
 *          catches any path that is not a pure bit copy. */
static inline float value_from_hash(uint64_t h, int mode) {
  if (mode == 0) {
    int q = (int)((h >> 52) & 0xFFF) - 2048;
    return (float)q * 0x1.0p-12f;
  }
  uint32_t b = (uint32_t)(h >> 32);
  if (((b >> 23) & 0xFF) == 0xFF) b &= ~(1u << 30);
  float f;
  memcpy(&f, &b, 4);
  return f;
}

static inline uint64_t row_hash(uint64_t s_val, int64_t t, int64_t row) {
  return sm64(sm64(s_val ^ (uint64_t)t) ^ (uint64_t)row);
}

EXPORT float flg_value(uint64_t s_val, int64_t t, int64_t row, int64_t col, int mode) {
  return value_from_hash(sm64(row_hash(s_val, t, row) ^ (uint64_t)col), mode);
}

/* Fill rows [row0, row0+nrows) of table t (dim d, row stride `ld` floats) into dst. */
EXPORT void flg_fill_table(uint64_t s_val, int64_t t, int64_t row0, int64_t nrows, int32_t d,
                           int64_t ld, int mode, float* dst, int nthreads) {
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(static, 4096) num_threads(nthreads)
#endif
  for (int64_t r = 0; r < nrows; ++r) {
    uint64_t hr = row_hash(s_val, t, row0 + r);
    float* o = dst + r * ld;
    for (int32_t c = 0; c < d; ++c) o[c] = value_from_hash(sm64(hr ^ (uint64_t)c), mode);
  }
}

/* ---- bounded Zipf by rejection-inversion ---------------------------------- */
typedef struct {
  double a, n, hIntX1, hIntN, sC;
} zipf_t;

static inline double H1(double y) { return fabs(y) > 1e-8 ? expm1(y) / y : 1.0 + y / 2.0 * (1.0 + y / 3.0 * (1.0 + y / 4.0)); }
static inline double H2(double y) { return fabs(y) > 1e-8 ? log1p(y) / y : 1.0 - y * (0.5 - y * (1.0 / 3.0 - y * 0.25)); }
static inline double zh(const zipf_t* z, double x) { return exp(-z->a * log(x)); }
static inline double zhI(const zipf_t* z, double x) {
  double lx = log(x);
  return H1((1.0 - z->a) * lx) * lx;
}
static inline double zhIinv(const zipf_t* z, double x) {
  double t = x * (1.0 - z->a);
  if (t < -1.0) t = -1.0;
  return exp(H2(t) * x);
}
static void zipf_init(zipf_t* z, double a, int64_t n) {
  z->a = a;
  z->n = (double)n;
  z->hIntX1 = zhI(z, 1.5) - 1.0;
  z->hIntN = zhI(z, (double)n + 0.5);
  z->sC = 2.0 - zhIinv(z, zhI(z, 2.5) - zh(z, 2.0));
}
/* rank in [1, n]; uniforms drawn from the counter stream q, q+1, ... */
static int64_t zipf_draw(const zipf_t* z, uint64_t q) {
  for (uint64_t k = 0;; ++k) {
    double u = u01(q + k);
    double uu = z->hIntN + u * (z->hIntX1 - z->hIntN);
    double x = zhIinv(z, uu);
    double kf = floor(x + 0.5);
    if (kf < 1.0) kf = 1.0;
    if (kf > z->n) kf = z->n;
    if (kf - x <= z->sC || uu >= zhI(z, kf + 0.5) - zh(z, kf)) return (int64_t)kf;
  }
}
EXPORT int64_t flg_zipf_rank(double a, int64_t n, uint64_t q) {
  zipf_t z;
  zipf_init(&z, a, n);
  return zipf_draw(&z, q);
}

/* ---- keyed rank -> row bijection ----------------------------------------- */
typedef struct {
  uint64_t mask, k1[3], k2[3];
  int f, sh;
  int64_t c;
} perm_t;

static int ceil_log2_i64(int64_t c) {
  int f = 0;
  while (f < 63 && ((int64_t)1 << f) < c) ++f;
  return f;
}
static void perm_init(perm_t* p, uint64_t s_perm, int64_t t, int64_t c) {
  int f = ceil_log2_i64(c);
  if (f < 1) f = 1;
  p->f = f;
  p->sh = (f + 1) / 2;
  p->mask = (f >= 64) ? ~0ULL : ((1ULL << f) - 1);
  p->c = c;
  for (int r = 0; r < 3; ++r) {
    p->k1[r] = sm64(s_perm ^ (uint64_t)(8 * t + r));
    p->k2[r] = sm64(s_perm ^ (uint64_t)(8 * t + r + 4));
  }
}
static inline uint64_t perm_round(const perm_t* p, uint64_t x) {
  for (int r = 0; r < 3; ++r) {
    x = (x + p->k1[r]) & p->mask;
    x = (x * (2 * p->k2[r] + 1)) & p->mask;
    x ^= x >> p->sh;
  }
  return x;
}
static inline int64_t perm_apply(const perm_t* p, int64_t rank0) {
  uint64_t x = perm_round(p, (uint64_t)rank0);
  while ((int64_t)x >= p->c) x = perm_round(p, x);
  return (int64_t)x;
}
EXPORT int64_t flg_perm(uint64_t s_perm, int64_t t, int64_t c, int64_t rank0) {
  perm_t p;
  perm_init(&p, s_perm, t, c);
  return perm_apply(&p, rank0);
}

/* ---- ID streams ----------------------------------------------------------- */
static inline uint64_t id_stream(uint64_t s_id, int64_t b, int64_t t, int64_t j) {
  return sm64(sm64(sm64(s_id ^ (uint64_t)b) ^ (uint64_t)t) ^ (uint64_t)j);
}

/* IDs of table t (cardinality c, skew a) for batch b, positions [j0, j0+n).
 * invalid_ppm > 0 replaces that many per million positions with an out-of-range
 * ID (negative or >= c) to exercise the invalid-ID contract. */
EXPORT void flg_gen_ids(uint64_t s_id, uint64_t s_perm, int64_t b, int64_t t, int64_t c, double a,
                        int64_t j0, int64_t n, int32_t invalid_ppm, int64_t* out, int nthreads) {
  zipf_t z;
  perm_t p;
  zipf_init(&z, a, c);
  perm_init(&p, s_perm, t, c);
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(static, 1024) num_threads(nthreads) if (n >= 16384)
#endif
  for (int64_t i = 0; i < n; ++i) {
    uint64_t q = id_stream(s_id, b, t, j0 + i);
    if (invalid_ppm > 0) {
      uint64_t h = sm64(q ^ 0xBADC0FFEE0DDF00DULL);
      if ((int64_t)(h % 1000000ULL) < invalid_ppm) {
        out[i] = ((h >> 20) & 1) ? -1 - (int64_t)((h >> 21) & 7) : c + (int64_t)((h >> 21) & 7);
        continue;
      }
    }
    int64_t r = zipf_draw(&z, q);
    out[i] = perm_apply(&p, r - 1);
  }
}

/* Bag lengths for a multi-hot table: L = 1 + floor(u * (2m - 1)), uniform on
 * {1, ..., 2m-1}, mean m. Writes CSR offsets[0..bags] (offsets[0] = 0). */
EXPORT int64_t flg_gen_bag_offsets(uint64_t s_bag, int64_t b, int64_t t, int32_t m, int64_t bag0,
                                   int64_t bags, int64_t* offsets) {
  offsets[0] = 0;
  for (int64_t i = 0; i < bags; ++i) {
    double u = u01(id_stream(s_bag, b, t, bag0 + i));
    int64_t L = 1 + (int64_t)floor(u * (double)(2 * m - 1));
    offsets[i + 1] = offsets[i] + L;
  }
  return offsets[bags];
}

/* IDs of a multi-hot table for bags [bag0, bag0+bags) given CSR offsets (offsets[0] = 0):
 * the k-th ID of global bag g uses ID-stream position g * 256 + k (bags are < 256 long),
 * so every ID is a pure function of (batch, table, bag, k) whatever the sharding. */
EXPORT void flg_gen_bag_ids(uint64_t s_id, uint64_t s_perm, int64_t b, int64_t t, int64_t c, double a,
                            int64_t bag0, int64_t bags, const int64_t* offsets, int32_t invalid_ppm,
                            int64_t* out, int nthreads) {
  zipf_t z;
  perm_t p;
  zipf_init(&z, a, c);
  perm_init(&p, s_perm, t, c);
#ifdef _OPENMP
  if (nthreads <= 0) nthreads = omp_get_max_threads();
#pragma omp parallel for schedule(static, 256) num_threads(nthreads) if (bags >= 4096)
#endif
  for (int64_t i = 0; i < bags; ++i) {
    for (int64_t k = offsets[i]; k < offsets[i + 1]; ++k) {
      uint64_t q = id_stream(s_id, b, t, (bag0 + i) * 256 + (k - offsets[i]));
      if (invalid_ppm > 0) {
        uint64_t h = sm64(q ^ 0xBADC0FFEE0DDF00DULL);
        if ((int64_t)(h % 1000000ULL) < invalid_ppm) {
          out[k] = ((h >> 20) & 1) ? -1 - (int64_t)((h >> 21) & 7) : c + (int64_t)((h >> 21) & 7);
          continue;
        }
      }
      out[k] = perm_apply(&p, zipf_draw(&z, q) - 1);
    }
  }
}
