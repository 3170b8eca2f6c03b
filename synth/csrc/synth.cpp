// synth.cpp — seeded synthetic INPUT generators shared by the oracle and the CUDA path.
//
// This file holds none of DGCL's arithmetic (no planning, no exchange, no reduction).  It only
// produces the inputs the paper's method consumes:
//   * an R-MAT power-law edge list shaped like the paper's datasets (Table 4),
//     because the datasets are not available offline;
//   * a balanced random vertex partition (stand-in for METIS);
//   * the required (remote-neighbour) list R_d of every GPU d, i.e. V^r_d of §4.1:
//     u is required by d iff some edge u->v has part[v] = d != part[u];
//   * hash-defined fp32 row values, so any element can be recomputed independently by the oracle.
//
// Every random draw is a counter-based splitmix64, so results do not depend on the thread count.
// Built with g++ -fopenmp into synth/_synth.so and called through ctypes (synth/graph.py).

#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <parallel/algorithm>
#include <vector>
#include <omp.h>
#include <cstdio>
#include <cstdlib>

namespace {

constexpr uint64_t kGolden = 0x9E3779B97F4A7C15ull;

inline uint64_t mix64(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
// First output of a splitmix64 stream seeded with x.
inline uint64_t sm64(uint64_t x) { return mix64(x + kGolden); }

struct KeyIdx {
  uint64_t key;
  uint64_t idx;
};

}  // namespace

extern "C" {

int synth_num_threads(void) { return omp_get_max_threads(); }

// Seeded Fisher-Yates permutation of [0, n): for i = n-1 .. 1, j = next() % (i+1), swap.
// next() is the sequential splitmix64 stream with state initialised to `seed`.
void synth_permutation(int64_t n, uint64_t seed, int64_t *out) {
  for (int64_t i = 0; i < n; ++i) out[i] = i;
  uint64_t state = seed;
  for (int64_t i = n - 1; i >= 1; --i) {
    state += kGolden;
    uint64_t r = mix64(state);
    int64_t j = (int64_t)(r % (uint64_t)(i + 1));
    std::swap(out[i], out[j]);
  }
}

// Balanced random partition: part[v] = perm[v] mod m.
void synth_partition(int64_t n, int32_t m, uint64_t seed, int32_t *part) {
  std::vector<int64_t> perm(n);
  synth_permutation(n, seed, perm.data());
  for (int64_t v = 0; v < n; ++v) part[v] = (int32_t)(perm[v] % m);
}

// One R-MAT edge attempt for counter `ctr`.  Level l (0 = most significant bit) draws a 16-bit
// uniform r from word l/4 of the attempt and picks the quadrant: r < ta -> (0,0); r < tab -> (0,1);
// r < tabc -> (1,0); else (1,1).  Returns UINT64_MAX for a rejected attempt (id >= n or self-loop).
static inline uint64_t rmat_attempt(uint64_t base, uint64_t ctr, int scale, int64_t n, uint32_t ta,
                                    uint32_t tab, uint32_t tabc) {
  uint64_t u = 0, v = 0;
  uint64_t w = 0;
  for (int l = 0; l < scale; ++l) {
    if ((l & 3) == 0) w = sm64(base + ctr * 8ull + (uint64_t)(l >> 2));
    uint32_t r = (uint32_t)((w >> (16 * (l & 3))) & 0xFFFFu);
    // quadrant: r < ta -> (0,0); r < tab -> (0,1); r < tabc -> (1,0); else (1,1)
    const uint64_t sb = r >= tab;
    const uint64_t db = (uint64_t)(r >= ta) ^ (uint64_t)(r >= tab) ^ (uint64_t)(r >= tabc);
    u = (u << 1) | sb;
    v = (v << 1) | db;
  }
  if ((int64_t)u >= n || (int64_t)v >= n || u == v) return UINT64_MAX;
  return (u << 32) | v;
}

// R-MAT directed edge list with exactly `e` distinct edges and no self-loops.
// Candidates are drawn in counter order; the first occurrence (lowest counter) of each key is
// accepted until e distinct keys exist.  Output is sorted by (src, dst).  Returns 0 on success.
int synth_rmat(int64_t n, int64_t e, uint64_t seed, double a, double b, double c, int32_t *src,
               int32_t *dst) {
  if (n < 2 || e < 0 || e > n * (n - 1)) return 1;
  int scale = 0;
  while ((1ll << scale) < n) ++scale;
  const uint32_t ta = (uint32_t)llround(a * 65536.0);
  const uint32_t tab = (uint32_t)llround((a + b) * 65536.0);
  const uint32_t tabc = (uint32_t)llround((a + b + c) * 65536.0);
  const uint64_t base = sm64(seed);
  std::vector<uint64_t> accepted;  // sorted unique keys
  accepted.reserve((size_t)e);
  uint64_t ctr = 0;
  while ((int64_t)accepted.size() < e) {
    const int64_t need = e - (int64_t)accepted.size();
    const int64_t batch = need + need / 4 + 4096;
    double tg = omp_get_wtime();
    // raw buffer: filled below in parallel (no serial zero-init / first-touch pass)
    KeyIdx *cand = static_cast<KeyIdx *>(std::malloc(sizeof(KeyIdx) * (size_t)batch));
    if (!cand) return 2;
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < batch; ++i) {
      cand[i].key = rmat_attempt(base, ctr + (uint64_t)i, scale, n, ta, tab, tabc);
      cand[i].idx = ctr + (uint64_t)i;
    }
    ctr += (uint64_t)batch;
    const bool verbose = std::getenv("SYNTH_VERBOSE") != nullptr;
    double t0 = omp_get_wtime();
    if (verbose) std::fprintf(stderr, "rmat: gen %.2fs\n", t0 - tg);
    __gnu_parallel::sort(cand, cand + batch, [](const KeyIdx &x, const KeyIdx &y) {
      return x.key != y.key ? x.key < y.key : x.idx < y.idx;
    });
    // keep first occurrence per key, not already accepted, valid
    std::vector<KeyIdx> fresh;
    fresh.reserve((size_t)batch);
    for (size_t i = 0; i < (size_t)batch; ++i) {
      if (cand[i].key == UINT64_MAX) break;  // sorted: invalids at the end
      if (i > 0 && cand[i].key == cand[i - 1].key) continue;
      if (std::binary_search(accepted.begin(), accepted.end(), cand[i].key)) continue;
      fresh.push_back(cand[i]);
    }
    std::free(cand);
    if (verbose) std::fprintf(stderr, "rmat: sort+filter %.2fs fresh=%zu need=%ld\n", omp_get_wtime() - t0, fresh.size(), (long)need);
    if ((int64_t)fresh.size() > need) {
      // keep the `need` lowest counters; `fresh` stays sorted by key
      std::vector<uint64_t> idx(fresh.size());
#pragma omp parallel for schedule(static)
      for (size_t i = 0; i < fresh.size(); ++i) idx[i] = fresh[i].idx;
      std::nth_element(idx.begin(), idx.begin() + (need - 1), idx.end());
      const uint64_t thr = idx[(size_t)(need - 1)];
      size_t w = 0;
      for (size_t i = 0; i < fresh.size(); ++i)
        if (fresh[i].idx <= thr) fresh[w++] = fresh[i];
      fresh.resize(w);
    }
    const size_t old = accepted.size();
    for (auto &f : fresh) accepted.push_back(f.key);
    std::inplace_merge(accepted.begin(), accepted.begin() + old, accepted.end());
    if (verbose) std::fprintf(stderr, "rmat: round done %.2fs\n", omp_get_wtime() - t0);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < e; ++i) {
    src[i] = (int32_t)(accepted[i] >> 32);
    dst[i] = (int32_t)(accepted[i] & 0xFFFFFFFFull);
  }
  return 0;
}

// Required (halo) lists.  R_d = { u : exists edge u->v with part[v] = d != part[u] }, ordered by
// ascending (owner part[u], u) — the harness's halo-row order (SURVEY §8(c) "Halo row order").
// Call with req_ids == NULL to get req_ptr (size m+1) only; then again with req_ids sized
// req_ptr[m].  Returns 0 on success.
int synth_required(int64_t n, int64_t e, const int32_t *src, const int32_t *dst, const int32_t *part,
                   int32_t m, int64_t *req_ptr, int64_t *req_ids) {
  std::vector<uint8_t> mark((size_t)n * (size_t)m, 0);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < e; ++i) {
    const int32_t u = src[i], v = dst[i];
    const int32_t pu = part[u], pv = part[v];
    if (pu != pv) mark[(size_t)u * m + pv] = 1;
  }
  // vertices bucketed by owner in ascending id
  std::vector<int64_t> optr(m + 1, 0);
  for (int64_t v = 0; v < n; ++v) optr[part[v] + 1]++;
  for (int d = 0; d < m; ++d) optr[d + 1] += optr[d];
  std::vector<int64_t> byowner((size_t)n);
  {
    std::vector<int64_t> fill(optr.begin(), optr.end() - 1);
    for (int64_t v = 0; v < n; ++v) byowner[fill[part[v]]++] = v;
  }
  std::vector<int64_t> cnt(m, 0);
#pragma omp parallel for schedule(static)
  for (int d = 0; d < m; ++d) {
    int64_t c = 0;
    for (int64_t i = 0; i < n; ++i) c += mark[(size_t)byowner[i] * m + d];
    cnt[d] = c;
  }
  req_ptr[0] = 0;
  for (int d = 0; d < m; ++d) req_ptr[d + 1] = req_ptr[d] + cnt[d];
  if (!req_ids) return 0;
#pragma omp parallel for schedule(static)
  for (int d = 0; d < m; ++d) {
    int64_t o = req_ptr[d];
    for (int64_t i = 0; i < n; ++i) {
      const int64_t u = byowner[i];
      if (mark[(size_t)u * m + d]) req_ids[o++] = u;
    }
  }
  return 0;
}

// Hash-defined fp32 values.  Row r of `out` (pitch elements apart) holds value(key_r, col) for
// col < dim, with key_r = keys[r] (or r when keys == NULL); padding columns are set to 0.
//   x = seed*K0 ^ stream*K3 ^ key*K1 ^ col*K2  (mod 2^64),  h = sm64(x)
//   mode 0 "uniform": ((h >> 40) * 2^-23) - 1       in [-1, 1), 24-bit grid, exact in fp32
//   mode 1 "ones":    1.0
//   mode 2 "int":     (h >> 60) - 8                 integers in [-8, 7]
//   mode 3 "bits":    raw uint32 (h >> 32)          (forward bit-copy tests only)
void synth_fill(float *out, int64_t rows, int64_t pitch, int64_t dim, const int64_t *keys,
                uint64_t seed, uint64_t stream, int32_t mode) {
  const uint64_t K0 = 0x9E3779B97F4A7C15ull, K1 = 0xD1B54A32D192ED03ull,
                 K2 = 0xABC98388FB8FAC03ull, K3 = 0xC2B2AE3D27D4EB4Full;
#pragma omp parallel for schedule(static)
  for (int64_t r = 0; r < rows; ++r) {
    const uint64_t key = keys ? (uint64_t)keys[r] : (uint64_t)r;
    const uint64_t xr = seed * K0 ^ stream * K3 ^ key * K1;
    float *row = out + r * pitch;
    for (int64_t col = 0; col < dim; ++col) {
      const uint64_t h = sm64(xr ^ ((uint64_t)col * K2));
      float v;
      if (mode == 0) {
        v = (float)((double)(h >> 40) * (1.0 / 8388608.0) - 1.0);
      } else if (mode == 1) {
        v = 1.0f;
      } else if (mode == 2) {
        v = (float)((int64_t)(h >> 60) - 8);
      } else {
        uint32_t bits = (uint32_t)(h >> 32);
        std::memcpy(&v, &bits, 4);
      }
      row[col] = v;
    }
    for (int64_t col = dim; col < pitch; ++col) row[col] = 0.0f;
  }
}

}  // extern "C"
