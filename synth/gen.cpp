// synth/gen.cpp — seeded synthetic inputs shared by the oracle and the CUDA path.
//
// This module holds NO arithmetic of the GNN-RDM method: it only draws graphs,
// features, labels and initial weights.  The recipe (DESIGN.md "Input recipe",
// SURVEY.md §8(d) "Generator"):
//   * R-MAT (Graph500 a,b,c,d = 0.57,0.19,0.19,0.05) over ids < 2^ceil(log2 N),
//     ids >= N rejected, self edges dropped, undirected de-duplication keeping
//     the earliest draw, truncated to EXACTLY `n_edges` undirected edges,
//     seeded random vertex permutation (Graph500 practice), symmetrized and
//     exactly one self loop per vertex added:  nnz = 2*n_edges + N.
//     (Table V: Reddit 114,848,857 = 2*57,307,946 + 232,965.)
//   * values: the GCN fixture normalization  Â = D̃^{-1/2}(A+I)D̃^{-1/2}
//     ("graph normalization code in CAGNET"; reading R6 in
//     DESIGN.md), computed in fp64 and stored fp32.  This is input
//     preparation — the library treats CSR values as opaque.
//   * features/weights/labels: counter-based splitmix64 hashes, identical
//     wherever they are evaluated.
// Everything is a pure function of (shape, seed): bit-identical across runs
// and thread counts.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <vector>
#include <omp.h>

namespace {

inline uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// Counter-based stream: value k of stream `s` under `seed`.
inline uint64_t ctr_hash(uint64_t seed, uint64_t s, uint64_t k) {
  return splitmix64(splitmix64(seed * 0x9E3779B97F4A7C15ull + s) ^ k);
}

// uniform in [0,1) with 24 random bits — exactly representable in fp32
inline double u24(uint64_t h) { return (double)(h >> 40) * (1.0 / 16777216.0); }

// Seeded Fisher-Yates permutation of [0, n).
void permutation(int64_t n, uint64_t seed, std::vector<int32_t>& perm) {
  perm.resize(n);
  for (int64_t i = 0; i < n; ++i) perm[i] = (int32_t)i;
  for (int64_t i = n - 1; i > 0; --i) {
    uint64_t h = ctr_hash(seed, 7, (uint64_t)i);
    int64_t j = (int64_t)(h % (uint64_t)(i + 1));
    std::swap(perm[i], perm[j]);
  }
}

struct Draw {
  int32_t u, v;  // u < v after canonicalisation
  int64_t k;     // draw index (earliest wins on duplicates)
};

}  // namespace

extern "C" {

uint64_t synth_splitmix64(uint64_t x) { return splitmix64(x); }

// R-MAT graph as symmetric CSR with self loops; see header comment.
// rowptr[n+1] (int64), col[nnz] (int32, sorted ascending within each row),
// val[nnz] (fp32, normalized).  nnz must equal 2*n_edges + n.
// Returns 0 on success, -1 if the draw budget could not produce n_edges
// unique edges, -2 on bad arguments.
int synth_rmat_csr(int64_t n, int64_t n_edges, uint64_t seed, double a, double b, double c,
                   int permute, int normalize, int64_t* rowptr, int32_t* col, float* val) {
  if (n <= 0 || n_edges < 0 || n > (int64_t)INT32_MAX) return -2;
  if (n_edges > n * (n - 1) / 2) return -2;
  int scale = 0;
  while ((int64_t(1) << scale) < n) ++scale;
  const double ab = a + b, abc = a + b + c;

  std::vector<int32_t> perm;
  if (permute) permutation(n, seed ^ 0x5eed5eedull, perm);

  // Draw in batches until the unique count reaches n_edges.
  std::vector<Draw> draws;
  int64_t next_k = 0;
  int64_t unique = 0;
  std::vector<Draw> uniq;
  int rounds = 0;
  while (true) {
    int64_t want = n_edges - unique;
    int64_t batch = std::max<int64_t>(1024, want + want / 4 + 64);
    if (rounds > 0) batch = std::max<int64_t>(batch, (next_k) / 8);
    size_t base = draws.size();
    draws.resize(base + batch);
#pragma omp parallel for schedule(static)
    for (int64_t t = 0; t < batch; ++t) {
      int64_t k = next_k + t;
      int64_t u = 0, v = 0;
      uint64_t h = 0;
      for (int lvl = 0; lvl < scale; ++lvl) {
        if ((lvl & 1) == 0) h = ctr_hash(seed, 1, (uint64_t)k * 64 + (uint64_t)(lvl >> 1));
        uint32_t bits = (lvl & 1) ? (uint32_t)(h >> 32) : (uint32_t)h;
        double r = (double)bits * (1.0 / 4294967296.0);
        int bu, bv;
        if (r < a) { bu = 0; bv = 0; }
        else if (r < ab) { bu = 0; bv = 1; }
        else if (r < abc) { bu = 1; bv = 0; }
        else { bu = 1; bv = 1; }
        u = 2 * u + bu;
        v = 2 * v + bv;
      }
      Draw d;
      d.k = k;
      if (u >= n || v >= n || u == v) { d.u = -1; d.v = -1; }
      else {
        int32_t pu = permute ? perm[u] : (int32_t)u;
        int32_t pv = permute ? perm[v] : (int32_t)v;
        d.u = std::min(pu, pv);
        d.v = std::max(pu, pv);
      }
      draws[base + t] = d;
    }
    next_k += batch;
    // de-duplicate: sort by (u, v, k), keep first of each (u, v)
    std::vector<Draw> all;
    all.reserve(uniq.size() + batch);
    all.insert(all.end(), uniq.begin(), uniq.end());
    for (size_t t = base; t < draws.size(); ++t)
      if (draws[t].u >= 0) all.push_back(draws[t]);
    draws.clear();
    // counting sort by u, then sort each bucket by (v, k)
    std::vector<int64_t> cnt(n + 1, 0);
    for (const Draw& d : all) cnt[d.u + 1]++;
    for (int64_t i = 0; i < n; ++i) cnt[i + 1] += cnt[i];
    std::vector<Draw> sorted(all.size());
    {
      std::vector<int64_t> pos(cnt.begin(), cnt.end() - 1);
      for (const Draw& d : all) sorted[pos[d.u]++] = d;
    }
    all.clear();
    all.shrink_to_fit();
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = 0; i < n; ++i) {
      std::sort(sorted.begin() + cnt[i], sorted.begin() + cnt[i + 1],
                [](const Draw& x, const Draw& y) { return x.v != y.v ? x.v < y.v : x.k < y.k; });
    }
    uniq.clear();
    for (size_t t = 0; t < sorted.size(); ++t) {
      if (t > 0 && sorted[t].u == sorted[t - 1].u && sorted[t].v == sorted[t - 1].v) continue;
      uniq.push_back(sorted[t]);
    }
    unique = (int64_t)uniq.size();
    ++rounds;
    if (unique >= n_edges) break;
    if (rounds > 64) return -1;
  }
  // keep the n_edges earliest unique draws
  if (unique > n_edges) {
    std::vector<int64_t> ks(uniq.size());
    for (size_t t = 0; t < uniq.size(); ++t) ks[t] = uniq[t].k;
    std::nth_element(ks.begin(), ks.begin() + (n_edges - 1), ks.end());
    int64_t kth = ks[n_edges - 1];  // k values are distinct
    std::vector<Draw> kept;
    kept.reserve(n_edges);
    for (const Draw& d : uniq)
      if (d.k <= kth) kept.push_back(d);
    uniq.swap(kept);
  }
  // symmetric CSR with self loops
  std::vector<int64_t> deg(n, 1);
  for (const Draw& d : uniq) { deg[d.u]++; deg[d.v]++; }
  rowptr[0] = 0;
  for (int64_t i = 0; i < n; ++i) rowptr[i + 1] = rowptr[i] + deg[i];
  {
    std::vector<int64_t> pos(rowptr, rowptr + n);
    for (int64_t i = 0; i < n; ++i) col[pos[i]++] = (int32_t)i;
    for (const Draw& d : uniq) {
      col[pos[d.u]++] = d.v;
      col[pos[d.v]++] = d.u;
    }
  }
#pragma omp parallel for schedule(dynamic, 256)
  for (int64_t i = 0; i < n; ++i) std::sort(col + rowptr[i], col + rowptr[i + 1]);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t i = 0; i < n; ++i) {
    double di = (double)(rowptr[i + 1] - rowptr[i]);
    for (int64_t j = rowptr[i]; j < rowptr[i + 1]; ++j) {
      if (normalize) {
        int32_t c2 = col[j];
        double dj = (double)(rowptr[c2 + 1] - rowptr[c2]);
        val[j] = (float)(1.0 / std::sqrt(di * dj));
      } else {
        val[j] = 1.0f;
      }
    }
  }
  return 0;
}

// Dense features: H0[i,j] = u24(hash(seed, i*f + j)) * 2 - 1 — exactly
// representable fp32 in [-1, 1).
void synth_features(int64_t n, int64_t f, uint64_t seed, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    for (int64_t j = 0; j < f; ++j)
      out[i * f + j] = (float)(u24(ctr_hash(seed, 2, (uint64_t)(i * f + j))) * 2.0 - 1.0);
}

// Rows [lo, hi) of the same features (one rank's row slice of a matrix too
// large to draw whole on the host).
void synth_features_rows(int64_t lo, int64_t hi, int64_t f, uint64_t seed, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = lo; i < hi; ++i)
    for (int64_t j = 0; j < f; ++j)
      out[(i - lo) * f + j] = (float)(u24(ctr_hash(seed, 2, (uint64_t)(i * f + j))) * 2.0 - 1.0);
}

// Glorot-uniform W (fin x fout, row-major): U[-s, s), s = sqrt(6/(fin+fout)).
void synth_glorot(int64_t fin, int64_t fout, uint64_t seed, float* out) {
  double s = std::sqrt(6.0 / (double)(fin + fout));
  for (int64_t i = 0; i < fin * fout; ++i)
    out[i] = (float)((u24(ctr_hash(seed, 3, (uint64_t)i)) * 2.0 - 1.0) * s);
}

// Labels in [0, C).
void synth_labels(int64_t n, int64_t C, uint64_t seed, int32_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) out[i] = (int32_t)(ctr_hash(seed, 4, (uint64_t)i) % (uint64_t)C);
}

// Labels of rows [lo, hi).
void synth_labels_rows(int64_t lo, int64_t hi, int64_t C, uint64_t seed, int32_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = lo; i < hi; ++i) out[i - lo] = (int32_t)(ctr_hash(seed, 4, (uint64_t)i) % (uint64_t)C);
}

// Train mask with a given keep fraction (1.0 -> all ones).
void synth_mask(int64_t n, double frac, uint64_t seed, uint8_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    out[i] = frac >= 1.0 ? 1 : (u24(ctr_hash(seed, 5, (uint64_t)i)) < frac ? 1 : 0);
}

int synth_num_threads(void) { return omp_get_max_threads(); }

}  // extern "C"
