// cpu_gather_probe.c — how fast can host threads gather random embedding rows?
//
// Measurement tool only (not product code).  Question: the GPU's zero-copy reads of
// random host rows are capped at ~80 M rows/s beyond a ~1 GiB span (profiles/
// hostlink_*_r01.json: IOMMU translation bound).  Host cores see no such cap; if T
// threads gather U random rows of a multi-GiB table into a contiguous pinned staging
// buffer faster than the GPU can fetch them, a CPU-assisted miss path can pay.
//
// usage: cpu_gather_probe SPAN_GIB ROW_BYTES   -> one JSON line
#define _GNU_SOURCE
#include <pthread.h>
#include <stdatomic.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <sys/mman.h>
#include <time.h>
#include <unistd.h>

static uint64_t sm64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
static double now(void) {
  struct timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return ts.tv_sec + 1e-9 * ts.tv_nsec;
}

typedef struct {
  const char* src;
  char* dst;
  const uint64_t* rows;
  int64_t n;
  int row;
  int tid, nt;
  _Atomic int* go;
  _Atomic int* done;
  int rounds;
} Arg;

static void gather(const Arg* a) {
  const int64_t per = (a->n + a->nt - 1) / a->nt;
  const int64_t lo = a->tid * per, hi = lo + per < a->n ? lo + per : a->n;
  const int PF = 16;
  for (int64_t i = lo; i < hi; ++i) {
    if (i + PF < hi) {
      const char* p = a->src + a->rows[i + PF] * (uint64_t)a->row;
      for (int c = 0; c < a->row; c += 64) __builtin_prefetch(p + c, 0, 0);
    }
    memcpy(a->dst + i * (int64_t)a->row, a->src + a->rows[i] * (uint64_t)a->row, a->row);
  }
}

static void* worker(void* p) {
  Arg* a = (Arg*)p;
  for (int r = 1; r <= a->rounds; ++r) {
    while (atomic_load_explicit(a->go, memory_order_acquire) < r) {
    }
    gather(a);
    atomic_fetch_add_explicit(a->done, 1, memory_order_acq_rel);
  }
  return NULL;
}

int main(int argc, char** argv) {
  const double span_gib = argc > 1 ? atof(argv[1]) : 8.0;
  const int row = argc > 2 ? atoi(argv[2]) : 256;
  const uint64_t bytes = (uint64_t)(span_gib * (1ull << 30));
  char* src = mmap(NULL, bytes, PROT_READ | PROT_WRITE, MAP_PRIVATE | MAP_ANONYMOUS, -1, 0);
  if (src == MAP_FAILED) return 1;
  madvise(src, bytes, MADV_HUGEPAGE);
  for (uint64_t o = 0; o < bytes; o += 4096) src[o] = (char)o;
  const uint64_t nrows = bytes / row;
  const int64_t maxn = 1 << 17;
  char* dst = aligned_alloc(4096, (size_t)maxn * row);
  uint64_t* rows = malloc(sizeof(uint64_t) * maxn);
  memset(dst, 0, (size_t)maxn * row);
  printf("{\"span_gib\": %.1f, \"row\": %d, \"ncpu\": %ld", span_gib, row, sysconf(_SC_NPROCESSORS_ONLN));
  const int ts[] = {1, 2, 4, 8, 12, 16};
  const int64_t ns[] = {8192, 32768, 131072};
  for (int ti = 0; ti < 6; ++ti) {
    const int nt = ts[ti];
    if (nt > sysconf(_SC_NPROCESSORS_ONLN)) break;
    for (int ni = 0; ni < 3; ++ni) {
      const int64_t n = ns[ni];
      const int rounds = 20;
      _Atomic int go = 0, done = 0;
      pthread_t th[16];
      Arg args[16];
      for (int t = 0; t < nt; ++t) {
        args[t] = (Arg){src, dst, rows, n, row, t, nt, &go, &done, rounds};
        pthread_create(&th[t], NULL, worker, &args[t]);
      }
      double best = 1e9, sum = 0;
      for (int r = 1; r <= rounds; ++r) {
        for (int64_t i = 0; i < n; ++i) rows[i] = sm64(((uint64_t)r << 40) ^ ((uint64_t)nt << 32) ^ i) % nrows;
        const double t0 = now();
        atomic_store_explicit(&go, r, memory_order_release);
        while (atomic_load_explicit(&done, memory_order_acquire) < r * nt) {
        }
        const double dt = now() - t0;
        if (r > 2) { sum += dt; if (dt < best) best = dt; }
      }
      for (int t = 0; t < nt; ++t) pthread_join(th[t], NULL);
      const double avg = sum / (rounds - 2);
      printf(", \"t%d_n%ld_us\": %.1f, \"t%d_n%ld_gbs\": %.2f", nt, (long)n, avg * 1e6, nt, (long)n,
             n * (double)row / avg / 1e9);
      fflush(stdout);
    }
  }
  printf("}\n");
  return 0;
}
