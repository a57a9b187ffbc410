// saint.cu — GraphSAINT-RDM sampler (§III-F, §V-C).
//
// Every rank draws the same subgraph from a shared seed (L173: "a random
// generated seed can be passed to all processes and each process can
// generate its sparse mask individually"), so sampling needs no
// communication; the subgraph is then trained with the ordinary RDM executor
// (L388 "each subgraph is parallelized using our RDM scheme").
//
// Device pipeline per subgraph (readings R31-R34, rdm.h):
//   walk_kernel      one thread per root: counter-based random walk
//   mark_kernel      flag[v] = 1 for every visited vertex
//   cub scan         map[v] = exclusive prefix of flag (new id of v)
//   compact_kernel   nodes[map[v]] = v (ascending), n_sub
//   rowseg/segrow    cut every sampled row's original list into 1024-entry
//                    segments (entry-parallel: hub rows do not serialise)
//   count_kernel     warp per segment: kept entries; d_i, Σ d_i (integer atomics)
//   cub scans        rowptr_s = prefix of d; segment output offsets
//   fill_kernel      warp per segment: col_s = map[u] in the original row order,
//                    val_s = (float)(1 / sqrt((double) d_i d_j))
// then the host builds the row bins from rowptr_s (one D2H copy, sharing its
// sync with the hub-core histogram when a core is built).
#include <cub/cub.cuh>

#include <algorithm>
#include <cmath>
#include <functional>
#include <vector>

#include "internal.h"

namespace rdm {
namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

uint64_t splitmix64_host(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void walk_kernel(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                            int64_t N, int64_t roots, int h, uint64_t key,
                            int32_t* __restrict__ visits) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= roots) return;
  const uint64_t base = (uint64_t)i << 8;
  int64_t v = (int64_t)(splitmix64(key ^ base) % (uint64_t)N);
  int32_t* out = visits + i * (h + 1);
  out[0] = (int32_t)v;
  for (int j = 1; j <= h; ++j) {
    const int64_t b = __ldg(rowptr + v), deg = __ldg(rowptr + v + 1) - b;
    if (deg > 0) v = __ldg(col + b + (int64_t)(splitmix64(key ^ (base | (uint64_t)j)) % (uint64_t)deg));
    out[j] = (int32_t)v;
  }
}

__global__ void mark_kernel(const int32_t* __restrict__ visits, int64_t count, int32_t* __restrict__ flag) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
       i += (int64_t)gridDim.x * blockDim.x)
    flag[visits[i]] = 1;
}

// nodes[map[v]] = v; scal[0] = n_sub
__global__ void compact_kernel(const int32_t* __restrict__ flag, const int32_t* __restrict__ map,
                               int64_t N, int32_t* __restrict__ nodes, unsigned long long* scal) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < N;
       v += (int64_t)gridDim.x * blockDim.x) {
    if (flag[v]) nodes[map[v]] = (int32_t)v;
    if (v == N - 1) scal[0] = (unsigned long long)(map[v] + flag[v]);
  }
}

// Every pass over adjacency entries is entry-parallel: each row's list (of
// the full graph for the sampled rows — random walks favour hubs, rows of
// 10^4-10^5 entries — or of the subgraph) is cut into kSeg-entry segments,
// one warp per segment, so a hub row does not serialise on one warp.
constexpr int kSeg = 1024;
constexpr int kMaxBuckets = 160;   // hub-core histogram: kmax <= 20480 in 128-buckets

// Row lengths for the segment tables: rows i < n of `rowptr`, through
// `nodes` (rows of the full graph) when given.  n from the device (scal[0])
// when `scal` is given, else n_host.
__device__ __forceinline__ int64_t seg_n(const unsigned long long* scal, int64_t n_host) {
  return scal ? (int64_t)scal[0] : n_host;
}

// nseg[i] = segments of row i, for i <= n_cap (0 beyond n)
__global__ void rowseg_kernel(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ nodes,
                              int64_t n_cap, const unsigned long long* scal, int64_t n_host,
                              int32_t* __restrict__ nseg) {
  const int64_t n = seg_n(scal, n_host);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= n_cap;
       i += (int64_t)gridDim.x * blockDim.x) {
    int32_t c = 0;
    if (i < n) {
      const int64_t v = nodes ? nodes[i] : i;
      c = (int32_t)((rowptr[v + 1] - rowptr[v] + kSeg - 1) / kSeg);
    }
    nseg[i] = c;
  }
}

__global__ void segrow_kernel(const int32_t* __restrict__ nseg, const int32_t* __restrict__ segoff,
                              const unsigned long long* scal, int64_t n_host,
                              int32_t* __restrict__ seg_row) {
  const int64_t n = seg_n(scal, n_host);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    for (int32_t k = 0; k < nseg[i]; ++k) seg_row[segoff[i] + k] = (int32_t)i;
}

struct Seg {     // segment sg of row i covers entries [b, end) of the row list
  int32_t i;
  int64_t b, end;
};
__device__ __forceinline__ Seg seg_of(int64_t sg, const int32_t* seg_row, const int32_t* segoff,
                                      const int64_t* rowptr, const int32_t* nodes) {
  Seg s;
  s.i = seg_row[sg];
  const int64_t v = nodes ? nodes[s.i] : s.i;
  const int64_t e = rowptr[v + 1];
  s.b = rowptr[v] + (sg - segoff[s.i]) * kSeg;
  s.end = s.b + kSeg < e ? s.b + kSeg : e;
  return s;
}

// warp per segment: kept entries c_s; d_i += c_s; scal[1] += c_s
__global__ void count_kernel(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                             const int32_t* __restrict__ flag, const int32_t* __restrict__ nodes,
                             const int32_t* __restrict__ seg_row, const int32_t* __restrict__ segoff,
                             int64_t n_cap, int64_t* __restrict__ cnt,
                             unsigned long long* __restrict__ deg, unsigned long long* scal) {
  const int lane = threadIdx.x & 31;
  const int64_t nsegs = segoff[n_cap];
  for (int64_t sg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; sg < nsegs;
       sg += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const Seg q = seg_of(sg, seg_row, segoff, rowptr, nodes);
    int c = 0;
    // 4 chunks of 32 entries per step: the column loads, then the flag
    // lookups, all independent (memory-level parallelism)
    for (int64_t k = q.b + lane; k < q.end; k += 128) {
      int32_t cc[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) cc[u] = (k + 32 * u < q.end) ? __ldg(col + k + 32 * u) : -1;
#pragma unroll
      for (int u = 0; u < 4; ++u) c += (cc[u] >= 0 && flag[cc[u]]) ? 1 : 0;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if (lane == 0) {
      cnt[sg] = c;
      if (c) {
        atomicAdd(deg + q.i, (unsigned long long)c);
        atomicAdd(scal + 1, (unsigned long long)c);
      }
    }
  }
}

// Per-warp-step histogram update: one shared atomic per distinct bucket.
__device__ __forceinline__ void bucket_add(unsigned* sb, int b, int lane) {
  const unsigned same = __match_any_sync(0xffffffffu, b);
  if (b >= 0 && lane == __ffs(same) - 1) atomicAdd(&sb[b], (unsigned)__popc(same));
}
__device__ __forceinline__ void bucket_flush(unsigned* sb, unsigned long long* bucket) {
  __syncthreads();
  for (int b = threadIdx.x; b < kMaxBuckets; b += blockDim.x)
    if (sb[b]) atomicAdd(bucket + b, (unsigned long long)sb[b]);
}

// warp per segment: kept entries in the original order at pos[s] onwards
__global__ void fill_kernel(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                            const int32_t* __restrict__ flag, const int32_t* __restrict__ map,
                            const int32_t* __restrict__ nodes, const int32_t* __restrict__ seg_row,
                            const int32_t* __restrict__ segoff, int64_t n_cap,
                            const unsigned long long* __restrict__ deg, const int64_t* __restrict__ pos,
                            int32_t* __restrict__ col_s, float* __restrict__ val_s) {
  const int lane = threadIdx.x & 31;
  const int64_t nsegs = segoff[n_cap];
  for (int64_t sg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; sg < nsegs;
       sg += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const Seg q = seg_of(sg, seg_row, segoff, rowptr, nodes);
    int64_t at0 = pos[sg];
    const double di = (double)deg[q.i];
    for (int64_t kb = q.b; kb < q.end; kb += 128) {
      // 4 chunks of 32 entries: loads batched, then compacted chunk by chunk
      // in the original order
      int32_t uu[4];
      bool kp[4];
#pragma unroll
      for (int c4 = 0; c4 < 4; ++c4) {
        const int64_t k = kb + 32 * c4 + lane;
        uu[c4] = k < q.end ? __ldg(col + k) : 0;
      }
#pragma unroll
      for (int c4 = 0; c4 < 4; ++c4) kp[c4] = (kb + 32 * c4 + lane < q.end) && flag[uu[c4]];
      // map / degree gathers of all 4 chunks issued before the compaction
      int32_t jj[4];
      unsigned long long dj[4];
#pragma unroll
      for (int c4 = 0; c4 < 4; ++c4) jj[c4] = kp[c4] ? map[uu[c4]] : 0;
#pragma unroll
      for (int c4 = 0; c4 < 4; ++c4) dj[c4] = kp[c4] ? deg[jj[c4]] : 1ull;
#pragma unroll
      for (int c4 = 0; c4 < 4; ++c4) {
        if (kb + 32 * c4 >= q.end) break;
        const unsigned m = __ballot_sync(0xffffffffu, kp[c4]);
        if (kp[c4]) {
          const int64_t at = at0 + __popc(m & ((1u << lane) - 1u));
          col_s[at] = jj[c4];
          val_s[at] = (float)(1.0 / sqrt(di * (double)dj[c4]));
        }
        at0 += __popc(m);
      }
    }
  }
}

// ---- dense hub core of a subgraph (device-side twin of spmm.cu build_core):
// degree-rank the vertices (stable, descending), histogram the entries by
// max(rank_i, rank_j) (fused into fill_kernel), pick K with the shared rule
// (choose_core_K), move the K x K block of the top-K vertices into a dense
// matrix and keep the rest as a residual CSR in the original order.
// Random-walk subgraphs are hub-heavy: for the Reddit-shaped config the top
// 12k of ~25k vertices hold ~88 % of the entries at ~20 % density.
__global__ void deg_key_kernel(const unsigned long long* __restrict__ deg, int64_t n,
                               int32_t* __restrict__ key, int32_t* __restrict__ iota) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    key[i] = (int32_t)deg[i];
    iota[i] = (int32_t)i;
  }
}

__global__ void rank_kernel(const int32_t* __restrict__ order, int64_t n, int32_t* __restrict__ rank) {
  for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n;
       k += (int64_t)gridDim.x * blockDim.x)
    rank[order[k]] = (int32_t)k;
}

// Histogram for the core size: entries by max(rank_i, rank_j) in 128-buckets
// below kmax, over the rows i ≡ 0 (mod 8) (a deterministic 1/8 sample; the
// size is a cost heuristic, the product is exact for any K).
__global__ void hist_kernel(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                            const int32_t* __restrict__ rank, const int32_t* __restrict__ seg_row,
                            const int32_t* __restrict__ segoff, int64_t n, int64_t kmax,
                            unsigned long long* __restrict__ bucket) {
  __shared__ unsigned sb[kMaxBuckets];
  for (int b = threadIdx.x; b < kMaxBuckets; b += blockDim.x) sb[b] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t nsegs = segoff[n];
  for (int64_t sg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; sg < nsegs;
       sg += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const int32_t i = seg_row[sg];
    if (i & 7) continue;                       // warp-uniform
    const Seg q = seg_of(sg, seg_row, segoff, rp, nullptr);
    const int32_t ri = rank[i];
    for (int64_t k0 = q.b; k0 < q.end; k0 += 128) {
      // 4 chunks of 32 entries: loads and rank lookups batched
      int32_t cc[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int64_t k = k0 + 32 * u + lane;
        cc[u] = k < q.end ? __ldg(col + k) : -1;
      }
      int bk[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        bk[u] = -1;
        if (cc[u] >= 0) {
          const int32_t mx = max(ri, rank[cc[u]]);
          if (mx < kmax) bk[u] = mx >> 7;
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) bucket_add(sb, bk[u], lane);
    }
  }
  bucket_flush(sb, bucket);
}

// CTA per hub (rank r < K): its dense row built in shared memory, then
// written whole (coalesced; zeros included, so no separate memset).  The
// col → rank gathers are batched kB per thread (independent loads in flight:
// hub rows of the dense subgraphs hold thousands of entries, and one
// dependent gather pair per iteration left the kernel latency-bound).
__global__ void core_rows_kernel(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                 const float* __restrict__ val, const int32_t* __restrict__ rank,
                                 const int32_t* __restrict__ order, int64_t K, float* __restrict__ dense) {
  constexpr int kB = 8;
  extern __shared__ float row[];
  for (int64_t r = blockIdx.x; r < K; r += gridDim.x) {
    for (int64_t c = threadIdx.x; c < K; c += blockDim.x) row[c] = 0.f;
    __syncthreads();
    const int32_t i = order[r];
    const int64_t e = rp[i + 1];
    for (int64_t k0 = rp[i] + threadIdx.x; k0 < e; k0 += (int64_t)kB * blockDim.x) {
      int32_t cj[kB];
      float vj[kB];
#pragma unroll
      for (int u = 0; u < kB; ++u) {
        const int64_t k = k0 + (int64_t)u * blockDim.x;
        cj[u] = k < e ? __ldg(col + k) : -1;
        vj[u] = k < e ? __ldg(val + k) : 0.f;
      }
      int32_t rj[kB];
#pragma unroll
      for (int u = 0; u < kB; ++u) rj[u] = cj[u] >= 0 ? __ldg(rank + cj[u]) : INT32_MAX;
#pragma unroll
      for (int u = 0; u < kB; ++u)
        if (rj[u] < K) row[rj[u]] = vj[u];   // CSR entries are distinct
    }
    __syncthreads();
    float4* out = reinterpret_cast<float4*>(dense + r * K);
    const float4* in = reinterpret_cast<const float4*>(row);
    for (int64_t c = threadIdx.x; c < K / 4; c += blockDim.x) out[c] = in[c];
    __syncthreads();
  }
}

// warp per subgraph segment: residual (non-core) entries counted
__global__ void resid_count_kernel(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                   const int32_t* __restrict__ rank, const int32_t* __restrict__ seg_row,
                                   const int32_t* __restrict__ segoff, int64_t n, int64_t K,
                                   int64_t* __restrict__ cnt) {
  const int lane = threadIdx.x & 31;
  const int64_t nsegs = segoff[n];
  for (int64_t sg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; sg < nsegs;
       sg += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const Seg q = seg_of(sg, seg_row, segoff, rp, nullptr);
    int c = 0;
    if (rank[q.i] >= K) {
      c = (int)(q.end - q.b);
    } else {
      for (int64_t k = q.b + lane; k < q.end; k += 128) {
        int32_t cc[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) cc[u] = (k + 32 * u < q.end) ? __ldg(col + k + 32 * u) : -1;
#pragma unroll
        for (int u = 0; u < 4; ++u) c += (cc[u] >= 0 && rank[cc[u]] >= K) ? 1 : 0;
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    }
    if (lane == 0) cnt[sg] = c;
  }
}

__global__ void resid_kernel(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                             const float* __restrict__ val, const int32_t* __restrict__ rank,
                             const int32_t* __restrict__ seg_row, const int32_t* __restrict__ segoff,
                             int64_t n, int64_t K, const int64_t* __restrict__ pos,
                             int32_t* __restrict__ rcol, float* __restrict__ rval) {
  const int lane = threadIdx.x & 31;
  const int64_t nsegs = segoff[n];
  for (int64_t sg = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; sg < nsegs;
       sg += ((int64_t)gridDim.x * blockDim.x) >> 5) {
    const Seg q = seg_of(sg, seg_row, segoff, rp, nullptr);
    const bool hub_i = rank[q.i] < K;
    int64_t at0 = pos[sg];
    for (int64_t kb = q.b; kb < q.end; kb += 128) {
      // 4 chunks of 32 entries: column / value loads and rank lookups batched,
      // then compacted chunk by chunk in the original order (as fill_kernel)
      int32_t cc[4];
      float vv[4];
      bool kp[4];
#pragma unroll
      for (int c4 = 0; c4 < 4; ++c4) {
        const int64_t k = kb + 32 * c4 + lane;
        cc[c4] = k < q.end ? __ldg(col + k) : 0;
        vv[c4] = k < q.end ? __ldg(val + k) : 0.f;
      }
#pragma unroll
      for (int c4 = 0; c4 < 4; ++c4)
        kp[c4] = (kb + 32 * c4 + lane < q.end) && !(hub_i && rank[cc[c4]] < K);
#pragma unroll
      for (int c4 = 0; c4 < 4; ++c4) {
        if (kb + 32 * c4 >= q.end) break;
        const unsigned m = __ballot_sync(0xffffffffu, kp[c4]);
        if (kp[c4]) {
          const int64_t at = at0 + __popc(m & ((1u << lane) - 1u));
          rcol[at] = cc[c4];
          rval[at] = vv[c4];
        }
        at0 += __popc(m);
      }
    }
  }
}

// residual rowptr from the segment offsets; hub ids / slots
__global__ void resid_rp_kernel(const int32_t* __restrict__ segoff, const int64_t* __restrict__ pos,
                                const int64_t* __restrict__ last_cnt, const int64_t* __restrict__ last_pos,
                                int64_t n, const int32_t* __restrict__ order,
                                const int32_t* __restrict__ rank, int64_t K, int64_t* __restrict__ rrp,
                                int32_t* __restrict__ hub_ids, int32_t* __restrict__ hub_slot) {
  const int64_t nsegs = segoff[n];
  const int64_t rnnz = *last_pos + *last_cnt;   // residual size: scan's last prefix + count
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= n;
       i += (int64_t)gridDim.x * blockDim.x) {
    rrp[i] = segoff[i] < nsegs ? pos[segoff[i]] : rnnz;
    if (i < n) {
      if (i < K) hub_ids[i] = order[i];
      hub_slot[i] = rank[i] < K ? rank[i] : -1;
    }
  }
}

__global__ void gather_kernel(const float* __restrict__ H, int64_t ldh, const int32_t* __restrict__ nodes,
                              int64_t row_lo, int64_t rows, int64_t col_lo, int64_t cols,
                              float* __restrict__ out, int64_t ldo) {
  const int64_t total = rows * cols;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total;
       t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = t / cols, c = t % cols;
    out[r * ldo + c] = __ldg(H + (int64_t)nodes[row_lo + r] * ldh + col_lo + c);
  }
}

__global__ void gather_labels_kernel(const int32_t* __restrict__ labels, const uint8_t* __restrict__ mask,
                                     const int32_t* __restrict__ nodes, int64_t row_lo, int64_t rows,
                                     int32_t* __restrict__ lab_out, uint8_t* __restrict__ mask_out) {
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < rows;
       r += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = nodes[row_lo + r];
    if (lab_out) lab_out[r] = labels[v];
    mask_out[r] = mask ? mask[v] : (uint8_t)1;
  }
}

unsigned grid_of(rdm_ctx* ctx, int64_t work, int per_block) {
  const int64_t b = ceil_div(std::max<int64_t>(work, 1), per_block);
  return (unsigned)std::min<int64_t>(b, (int64_t)ctx->num_sms * 16);
}

template <class In, class Out>
void scan(rdm_ctx* ctx, std::unique_ptr<DevBuf>& tmp, In* in, Out* out, int64_t count) {
  size_t t = 0;
  RDM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, t, in, out, (int)count, ctx->stream));
  void* w = ensure_ws(tmp, std::max<size_t>(t, 256));
  RDM_CUDA(cub::DeviceScan::ExclusiveSum(w, t, in, out, (int)count, ctx->stream));
}

// Core size bound for a subgraph of n vertices: 0 = no core considered.
// RDM_NO_CORE=1 disables; RDM_SAINT_CORE_K forces a size (tests).
int64_t core_kmax(int64_t n, int64_t nnz) {
  const char* off = getenv("RDM_NO_CORE");
  const char* force = getenv("RDM_SAINT_CORE_K");
  const bool forced = force && atoi(force) > 0;
  if ((off && atoi(off)) || nnz == 0 || (n < 4096 && !forced)) return 0;
  const int64_t kmax = std::min<int64_t>((forced ? n : n / 2) / 128 * 128, 128 * kMaxBuckets);
  return kmax >= (forced ? 128 : 1024) ? kmax : 0;
}

// Hub core of the current subgraph S, first half (needs S.n, S.nnz and the
// CSR of S, not its bins): ranks and the sampled histogram, whose copy into
// the pinned hb is issued here and waited for by the caller together with
// the rowptr of S (one host sync for both).
void build_core_sub(rdm_saint* s, Csr& S, int64_t kmax, const unsigned long long* deg,
                    unsigned long long* hb) {
  rdm_ctx* ctx = s->ctx;
  const int64_t n = S.n, nnz = S.nnz;
  const int64_t* rp = S.rowptr->as<int64_t>();
  const int32_t* col = S.col->as<int32_t>();
  // degree order (stable, descending) and ranks
  int32_t* keys = reinterpret_cast<int32_t*>(ensure_ws(s->core_tmp, (size_t)4 * n * sizeof(int32_t) + 256));
  int32_t* iota = keys + n;
  int32_t* keys_sorted = iota + n;
  int32_t* order = keys_sorted + n;
  int32_t* rank = reinterpret_cast<int32_t*>(ensure_ws(s->core_rank, n * sizeof(int32_t)));
  deg_key_kernel<<<grid_of(ctx, n, 256), 256, 0, ctx->stream>>>(deg, n, keys, iota);
  RDM_LAUNCHED(ctx);
  size_t tb = 0;
  RDM_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, keys, keys_sorted, iota, order, (int)n, 0,
                                                      32, ctx->stream));
  void* tmp = ensure_ws(s->tmp2, std::max<size_t>(tb, 256));
  RDM_CUDA(cub::DeviceRadixSort::SortPairsDescending(tmp, tb, keys, keys_sorted, iota, order, (int)n, 0, 32,
                                                      ctx->stream));
  rank_kernel<<<grid_of(ctx, n, 256), 256, 0, ctx->stream>>>(order, n, rank);
  RDM_LAUNCHED(ctx);
  // segment tables of S
  const int64_t seg_cap = n + nnz / kSeg + 1;
  int32_t* nseg = reinterpret_cast<int32_t*>(ensure_ws(s->core_seg, (2 * (n + 1) + seg_cap) * 4 + 16));
  int32_t* segoff = nseg + (n + 1);
  int32_t* seg_row = segoff + (n + 1);
  ensure_ws(s->core_cnt, 2 * seg_cap * sizeof(int64_t));   // sized here: the residual pass reuses it
  unsigned long long* bucket = reinterpret_cast<unsigned long long*>(ensure_ws(s->core_bucket, kMaxBuckets * 8));
  rowseg_kernel<<<grid_of(ctx, n + 1, 256), 256, 0, ctx->stream>>>(rp, nullptr, n, nullptr, n, nseg);
  RDM_LAUNCHED(ctx);
  scan(ctx, s->tmp, nseg, segoff, n + 1);
  segrow_kernel<<<grid_of(ctx, n, 256), 256, 0, ctx->stream>>>(nseg, segoff, nullptr, n, seg_row);
  RDM_LAUNCHED(ctx);
  RDM_CUDA(cudaMemsetAsync(bucket, 0, kMaxBuckets * 8, ctx->stream));
  hist_kernel<<<grid_of(ctx, seg_cap * 32, 256), 256, 0, ctx->stream>>>(rp, col, rank, seg_row, segoff, n, kmax,
                                                                         bucket);
  RDM_LAUNCHED(ctx);
  RDM_CUDA(cudaMemcpyAsync(hb, bucket, kMaxBuckets * 8, cudaMemcpyDeviceToHost, ctx->stream));
}

// Second half, after the host sync that delivered hb (shared with the rowptr
// of S): K, dense rows, residual CSR (+ its bins).  The workspaces are the
// ones the first half sized (ensure_ws keeps them).
void build_core_sub_finish(rdm_saint* s, Csr& S, int64_t kmax, const unsigned long long* hb) {
  rdm_ctx* ctx = s->ctx;
  const int64_t n = S.n, nnz = S.nnz;
  Core& c = S.core;
  const int64_t* rp = S.rowptr->as<int64_t>();
  const int32_t* col = S.col->as<int32_t>();
  const float* val = S.val->as<float>();
  int32_t* keys = reinterpret_cast<int32_t*>(ensure_ws(s->core_tmp, (size_t)4 * n * sizeof(int32_t) + 256));
  int32_t* order = keys + 3 * n;
  int32_t* rank = reinterpret_cast<int32_t*>(ensure_ws(s->core_rank, n * sizeof(int32_t)));
  const int64_t seg_cap = n + nnz / kSeg + 1;
  int32_t* nseg = reinterpret_cast<int32_t*>(ensure_ws(s->core_seg, (2 * (n + 1) + seg_cap) * 4 + 16));
  int32_t* segoff = nseg + (n + 1);
  int32_t* seg_row = segoff + (n + 1);
  int64_t* cnt = reinterpret_cast<int64_t*>(ensure_ws(s->core_cnt, 2 * seg_cap * sizeof(int64_t)));
  int64_t* pos = cnt + seg_cap;
  std::vector<int64_t> b64(kMaxBuckets);
  for (int b = 0; b < kMaxBuckets; ++b) b64[b] = (int64_t)hb[b] * 8;   // 1/8 row sample
  bool forced = false;
  const int64_t K = choose_core_K(b64.data(), kmax, getenv("RDM_SAINT_CORE_K"), &forced);
  if (!K) return;
  // dense rows of the hubs
  float* dense = ensure_ws(c.A, (size_t)K * K * sizeof(float));
  const int smem = (int)(K * sizeof(float));
  RDM_CUDA(cudaFuncSetAttribute(core_rows_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  int per_sm = 0;   // as many resident CTAs as the K-float row buffer allows
  RDM_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, core_rows_kernel, 256, smem));
  per_sm = std::max(per_sm, 1);
  core_rows_kernel<<<(unsigned)std::min<int64_t>(K, (int64_t)ctx->num_sms * per_sm), 256, smem, ctx->stream>>>(
      rp, col, val, rank, order, K, dense);
  RDM_LAUNCHED(ctx);
  // residual CSR: count, scan, fill in the original order
  RDM_CUDA(cudaMemsetAsync(cnt, 0, seg_cap * sizeof(int64_t), ctx->stream));
  resid_count_kernel<<<grid_of(ctx, seg_cap * 32, 256), 256, 0, ctx->stream>>>(rp, col, rank, seg_row, segoff,
                                                                                 n, K, cnt);
  RDM_LAUNCHED(ctx);
  scan(ctx, s->tmp, cnt, pos, seg_cap);
  if (!c.resid) c.resid.reset(new Csr());
  Csr& R = *c.resid;
  int64_t* rrp = reinterpret_cast<int64_t*>(ensure_ws(R.rowptr, (n + 1) * sizeof(int64_t)));
  // residual arrays sized by nnz (an upper bound: no host round trip for the
  // exact size; resid_rp_kernel reads it from the scan's last prefix + count,
  // and the host learns it with the residual rowptr)
  int32_t* rcol = reinterpret_cast<int32_t*>(ensure_ws(R.col, std::max<int64_t>(nnz, 1) * sizeof(int32_t)));
  float* rval = ensure_ws(R.val, std::max<int64_t>(nnz, 1) * sizeof(float));
  resid_kernel<<<grid_of(ctx, seg_cap * 32, 256), 256, 0, ctx->stream>>>(rp, col, val, rank, seg_row, segoff,
                                                                          n, K, pos, rcol, rval);
  RDM_LAUNCHED(ctx);
  int32_t* hub_ids = reinterpret_cast<int32_t*>(ensure_ws(c.hub_ids, K * sizeof(int32_t)));
  int32_t* hub_slot = reinterpret_cast<int32_t*>(ensure_ws(c.hub_slot, n * sizeof(int32_t)));
  resid_rp_kernel<<<grid_of(ctx, n + 1, 256), 256, 0, ctx->stream>>>(segoff, pos, cnt + seg_cap - 1,
                                                                       pos + seg_cap - 1, n, order, rank, K,
                                                                       rrp, hub_ids, hub_slot);
  RDM_LAUNCHED(ctx);
  int64_t* rrph = s->h_rrp.get<int64_t>(n + 1);
  RDM_CUDA(cudaMemcpyAsync(rrph, rrp, (n + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, ctx->stream));
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  const int64_t rnnz = rrph[n];
  R.n = n;
  R.nnz = rnnz;
  build_bins(ctx, R, rrph, false);
  c.K = K;
  c.nnz = nnz - rnnz;
  c.forced = forced;
}

template <class In, class Out>
size_t scan_temp_bytes(int64_t count) {
  size_t t = 0;
  RDM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, t, (In*)nullptr, (Out*)nullptr, (int)count, (cudaStream_t)0));
  return t;
}

// Bins of a CSR with at most `rows` rows and `nnz` entries (spmm.cu: light
// rows + 2048-entry segments of heavy rows) and their pinned staging.
void reserve_bins(Csr& C, int64_t rows, int64_t nnz) {
  const int64_t seg = nnz / 2048 + rows + 1;
  ensure_ws(C.light_rows, std::max<int64_t>(1, rows) * sizeof(int32_t));
  ensure_ws(C.seg_start, seg * (sizeof(int64_t) + sizeof(int32_t)));
  ensure_ws(C.heavy_rows, std::max<int64_t>(1, rows) * sizeof(int32_t));
  ensure_ws(C.heavy_seg, (rows + 1) * sizeof(int32_t));
  C.bins_stage.reserve((size_t)seg * 12 + (size_t)(3 * rows + 1) * 4 + 64);
}

// Every workspace of the sampler sized once at its bound, so that no step
// allocates (a regrowth inside a step was the cause of the step-time spikes):
// a subgraph has at most n_cap vertices and at most
//   nnz_bound = min(nnz(A), Σ of the n_cap largest degrees, n_cap²)
// entries; its hub core at most core_kmax(n_cap) hubs.
void reserve_bounds(rdm_saint* s) {
  rdm_ctx* ctx = s->ctx;
  const Csr& A = ctx->graph.A;
  const int64_t N = A.n, cap = s->n_cap;
  std::vector<int64_t> rp(N + 1);
  RDM_CUDA(cudaMemcpy(rp.data(), A.rowptr->ptr, (N + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost));
  std::vector<int64_t> deg(N);
  for (int64_t i = 0; i < N; ++i) deg[i] = rp[i + 1] - rp[i];
  if (cap < N) std::nth_element(deg.begin(), deg.begin() + cap, deg.end(), std::greater<int64_t>());
  int64_t top = 0;
  for (int64_t i = 0; i < cap; ++i) top += deg[i];
  const int64_t nnzb = std::max<int64_t>(1, std::min<int64_t>({A.nnz, top, cap * cap}));
  const int64_t seg_full = cap + A.nnz / kSeg + 1;
  const int64_t seg_sub = cap + nnzb / kSeg + 1;
  const int64_t kmax = core_kmax(cap, nnzb);
  s->nnz_bound = nnzb;
  for (int b = 0; b < 2; ++b) {
    Csr& S = s->bufs[b].A;
    ensure_ws(S.rowptr, (cap + 1) * sizeof(int64_t));
    ensure_ws(S.col, nnzb * sizeof(int32_t));
    ensure_ws(S.val, nnzb * sizeof(float));
    reserve_bins(S, cap, nnzb);
    ensure_ws(s->nodes_b[b], cap * sizeof(int32_t));
    if (kmax) {
      Core& c = S.core;
      ensure_ws(c.A, (size_t)kmax * kmax * sizeof(float));
      if (!c.resid) c.resid.reset(new Csr());
      Csr& R = *c.resid;
      ensure_ws(R.rowptr, (cap + 1) * sizeof(int64_t));
      ensure_ws(R.col, nnzb * sizeof(int32_t));
      ensure_ws(R.val, nnzb * sizeof(float));
      reserve_bins(R, cap, nnzb);
      ensure_ws(c.hub_ids, kmax * sizeof(int32_t));
      ensure_ws(c.hub_slot, cap * sizeof(int32_t));
    }
  }
  ensure_ws(s->core_tmp, (size_t)4 * cap * sizeof(int32_t) + 256);
  ensure_ws(s->core_rank, cap * sizeof(int32_t));
  ensure_ws(s->core_seg, (2 * (cap + 1) + seg_sub) * 4 + 16);
  ensure_ws(s->core_cnt, 2 * seg_sub * sizeof(int64_t));
  ensure_ws(s->core_bucket, kMaxBuckets * 8);
  size_t t = 256;
  t = std::max(t, scan_temp_bytes<int32_t, int32_t>(std::max<int64_t>(N, cap + 1)));
  t = std::max(t, scan_temp_bytes<unsigned long long, int64_t>(cap + 1));
  t = std::max(t, scan_temp_bytes<int64_t, int64_t>(std::max(seg_full, seg_sub)));
  ensure_ws(s->tmp, t);
  size_t tb = 0;
  RDM_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, (int32_t*)nullptr, (int32_t*)nullptr,
                                                      (int32_t*)nullptr, (int32_t*)nullptr, (int)cap, 0, 32,
                                                      (cudaStream_t)0));
  ensure_ws(s->tmp2, std::max<size_t>(tb, 256));
  s->h_rp.reserve((cap + 1) * sizeof(int64_t));
  s->h_rrp.reserve((cap + 1) * sizeof(int64_t));
  s->h_scal.reserve(4 * sizeof(unsigned long long));
  s->h_bucket.reserve(kMaxBuckets * sizeof(unsigned long long));
  s->reserved = true;
}

void sample(rdm_saint* s, int64_t it, int64_t* n_out, int64_t* nnz_out) {
  rdm_ctx* ctx = s->ctx;
  // the whole build runs on the sampler's stream (host round trips wait for
  // it only), into the buffer not in use by the subgraph being trained
  if (!s->sst) {
    // high priority: the host waits on this stream several times per subgraph,
    // so its short kernels go first whenever SMs free up between the
    // training kernels of the previous subgraph
    int lo = 0, hi = 0;
    RDM_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
    RDM_CUDA(cudaStreamCreateWithPriority(&s->sst, cudaStreamNonBlocking, hi));
    for (int b = 0; b < 2; ++b) {
      RDM_CUDA(cudaEventCreateWithFlags(&s->ev_done[b], cudaEventDisableTiming));
      RDM_CUDA(cudaEventCreateWithFlags(&s->ev_free[b], cudaEventDisableTiming));
    }
  }
  if (!s->reserved) reserve_bounds(s);
  const int b = s->iteration < 0 ? 0 : (s->cur ^ 1);
  struct OnStream {
    rdm_ctx* c; cudaStream_t m;
    ~OnStream() { c->stream = m; }
  } on{ctx, ctx->stream};
  // the previous sample (same workspaces) was issued on the sampler stream
  // already; the buffer must have been released by the executor
  if (s->freed[b]) RDM_CUDA(cudaStreamWaitEvent(s->sst, s->ev_free[b], 0));
  else RDM_CUDA(cudaStreamSynchronize(ctx->stream));   // never trained on: nothing to wait for but the setup
  ctx->stream = s->sst;
  Phase ph(ctx, RDM_PH_SAMPLE);
  const Csr& A = ctx->graph.A;
  const int64_t N = A.n, cap = s->n_cap;
  const int h = s->walk_len;
  const int64_t nv = s->roots * (h + 1);
  // segments of the sampled rows: at most one partial segment per row
  const int64_t seg_cap = cap + A.nnz / kSeg + 1;
  int32_t* visits = reinterpret_cast<int32_t*>(ensure_ws(s->visits, nv * sizeof(int32_t)));
  int32_t* flag = reinterpret_cast<int32_t*>(ensure_ws(s->flag, N * sizeof(int32_t)));
  int32_t* map = reinterpret_cast<int32_t*>(ensure_ws(s->map, N * sizeof(int32_t)));
  int32_t* nodes = reinterpret_cast<int32_t*>(ensure_ws(s->nodes_b[b], cap * sizeof(int32_t)));
  unsigned long long* deg = reinterpret_cast<unsigned long long*>(ensure_ws(s->deg, (cap + 1) * 8));
  // segment tables: nseg[cap+1] | segoff[cap+1] | seg_row[seg_cap] (int32); cnt | pos (int64)
  int32_t* nseg = reinterpret_cast<int32_t*>(ensure_ws(s->seg, (2 * (cap + 1) + seg_cap) * 4 + 16));
  int32_t* segoff = nseg + (cap + 1);
  int32_t* seg_row = segoff + (cap + 1);
  int64_t* cnt = reinterpret_cast<int64_t*>(ensure_ws(s->rps, 2 * seg_cap * sizeof(int64_t)));
  int64_t* pos = cnt + seg_cap;
  unsigned long long* scal = reinterpret_cast<unsigned long long*>(ensure_ws(s->scal, 64));

  const uint64_t key = splitmix64_host(s->seed + (uint64_t)it * 0x9E3779B97F4A7C15ull);
  RDM_CUDA(cudaMemsetAsync(flag, 0, N * sizeof(int32_t), ctx->stream));
  RDM_CUDA(cudaMemsetAsync(scal, 0, 64, ctx->stream));
  RDM_CUDA(cudaMemsetAsync(deg, 0, (cap + 1) * 8, ctx->stream));
  RDM_CUDA(cudaMemsetAsync(cnt, 0, seg_cap * 8, ctx->stream));
  walk_kernel<<<(unsigned)ceil_div(s->roots, 128), 128, 0, ctx->stream>>>(
      A.rowptr->as<int64_t>(), A.col->as<int32_t>(), N, s->roots, h, key, visits);
  RDM_LAUNCHED(ctx);
  mark_kernel<<<grid_of(ctx, nv, 256), 256, 0, ctx->stream>>>(visits, nv, flag);
  RDM_LAUNCHED(ctx);
  scan(ctx, s->tmp, flag, map, N);
  compact_kernel<<<grid_of(ctx, N, 256), 256, 0, ctx->stream>>>(flag, map, N, nodes, scal);
  RDM_LAUNCHED(ctx);
  rowseg_kernel<<<grid_of(ctx, cap + 1, 256), 256, 0, ctx->stream>>>(A.rowptr->as<int64_t>(), nodes, cap,
                                                                       scal, 0, nseg);
  RDM_LAUNCHED(ctx);
  scan(ctx, s->tmp, nseg, segoff, cap + 1);
  segrow_kernel<<<grid_of(ctx, cap, 256), 256, 0, ctx->stream>>>(nseg, segoff, scal, 0, seg_row);
  RDM_LAUNCHED(ctx);
  count_kernel<<<grid_of(ctx, seg_cap * 32, 256), 256, 0, ctx->stream>>>(
      A.rowptr->as<int64_t>(), A.col->as<int32_t>(), flag, nodes, seg_row, segoff, cap, cnt, deg, scal);
  RDM_LAUNCHED(ctx);
  unsigned long long* hs = s->h_scal.get<unsigned long long>(2);
  RDM_CUDA(cudaMemcpyAsync(hs, scal, 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost, ctx->stream));
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  const int64_t n = (int64_t)hs[0], nnz = (int64_t)hs[1];
  if (n > cap || nnz > s->nnz_bound) throw Error(RDM_ERR_STATE, "saint: subgraph larger than its bound");

  Graph& G = s->bufs[b];
  Csr& S = G.A;
  S.core.K = 0;
  S.core.nnz = 0;
  int64_t* rp = reinterpret_cast<int64_t*>(ensure_ws(S.rowptr, (cap + 1) * sizeof(int64_t)));
  int32_t* cs = reinterpret_cast<int32_t*>(ensure_ws(S.col, std::max<int64_t>(nnz, 1) * sizeof(int32_t)));
  float* vs = ensure_ws(S.val, std::max<int64_t>(nnz, 1) * sizeof(float));
  // rowptr_s: prefix of d (zero beyond n); segment output offsets: prefix of c
  scan(ctx, s->tmp, deg, rp, cap + 1);
  scan(ctx, s->tmp, cnt, pos, seg_cap);
  fill_kernel<<<grid_of(ctx, seg_cap * 32, 256), 256, 0, ctx->stream>>>(
      A.rowptr->as<int64_t>(), A.col->as<int32_t>(), flag, map, nodes, seg_row, segoff, cap, deg, pos,
      cs, vs);
  RDM_LAUNCHED(ctx);
  int64_t* rph = s->h_rp.get<int64_t>(n + 1);
  RDM_CUDA(cudaMemcpyAsync(rph, rp, (n + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, ctx->stream));
  S.n = n;
  S.nnz = nnz;
  // the hub core's ranks + histogram need the CSR of S, not its bins: issued
  // before the host waits, so that one sync brings back rowptr_s and the
  // histogram together
  const int64_t kmax = core_kmax(n, nnz);
  unsigned long long* hb = s->h_bucket.get<unsigned long long>(kMaxBuckets);
  if (kmax) build_core_sub(s, S, kmax, deg, hb);
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  // bins uploaded asynchronously on the sampler stream: their pinned staging is
  // rewritten only two samples later, after this stream has been synchronised
  build_bins(ctx, S, rph, false);
  if (kmax) build_core_sub_finish(s, S, kmax, hb);
  G.n = n;
  G.nnz = nnz;
  G.symmetric = true;
  RDM_CUDA(cudaEventRecord(s->ev_done[b], s->sst));
  s->freed[b] = false;
  s->cur = b;
  s->iteration = it;
  s->version++;
  *n_out = n;
  *nnz_out = nnz;
}

}  // namespace

void saint_gather(rdm_ctx* ctx, const float* H, int64_t ldh, const int32_t* nodes, int64_t row_lo,
                  int64_t rows, int64_t col_lo, int64_t cols, float* out, int64_t ldo) {
  if (rows * cols == 0) return;
  gather_kernel<<<grid_of(ctx, rows * cols, 256), 256, 0, ctx->stream>>>(H, ldh, nodes, row_lo, rows,
                                                                          col_lo, cols, out, ldo);
  RDM_LAUNCHED(ctx);
}

void saint_gather_labels(rdm_ctx* ctx, const int32_t* labels, const uint8_t* mask,
                         const int32_t* nodes, int64_t row_lo, int64_t rows, int32_t* lab_out,
                         uint8_t* mask_out) {
  if (rows == 0) return;
  gather_labels_kernel<<<grid_of(ctx, rows, 256), 256, 0, ctx->stream>>>(labels, mask, nodes, row_lo,
                                                                          rows, lab_out, mask_out);
  RDM_LAUNCHED(ctx);
}

}  // namespace rdm

using namespace rdm;

rdm_status rdm_guarded_call(rdm_ctx* ctx, void (*fn)(void*), void* arg);

extern "C" {

rdm_status rdm_saint_create(rdm_ctx* ctx, int64_t roots, int walk_len, uint64_t seed,
                            rdm_saint** out) {
  if (!ctx || !out || roots < 1 || walk_len < 0 || walk_len > 255) return RDM_ERR_ARG;
  if (!ctx->has_graph) {
    ctx->err = "rdm_saint_create: no graph (call rdm_set_graph)";
    return RDM_ERR_STATE;
  }
  if (!ctx->graph.symmetric) {
    ctx->err = "rdm_saint_create: the sampler needs a symmetric graph";
    return RDM_ERR_UNSUPPORTED;
  }
  if (ctx->graph.n < 1 || ctx->graph.n >= (int64_t)INT32_MAX) return RDM_ERR_ARG;
  auto* s = new rdm_saint();
  s->ctx = ctx;
  s->roots = roots;
  s->walk_len = walk_len;
  s->seed = seed;
  s->n_cap = std::min<int64_t>(ctx->graph.n, roots * (walk_len + 1));
  *out = s;
  return RDM_OK;
}

rdm_status rdm_saint_destroy(rdm_saint* s) {
  if (!s) return RDM_ERR_ARG;
  cudaSetDevice(s->ctx->device);
  cudaStreamSynchronize(s->ctx->stream);
  if (s->sst) {
    cudaStreamSynchronize(s->sst);
    cudaStreamDestroy(s->sst);
    for (int b = 0; b < 2; ++b) {
      cudaEventDestroy(s->ev_done[b]);
      cudaEventDestroy(s->ev_free[b]);
    }
  }
  delete s;
  release_retired();
  return RDM_OK;
}

namespace {
struct SampleArgs {
  rdm_saint* s;
  int64_t it;
  int64_t *n, *nnz;
};
}  // namespace

rdm_status rdm_saint_sample(rdm_saint* s, int64_t iteration, int64_t* n_sub, int64_t* nnz_sub) {
  if (!s || iteration < 0) return RDM_ERR_ARG;
  int64_t n = 0, nnz = 0;
  SampleArgs a{s, iteration, &n, &nnz};
  rdm_status st = rdm_guarded_call(
      s->ctx, [](void* p) {
        auto* q = static_cast<SampleArgs*>(p);
        sample(q->s, q->it, q->n, q->nnz);
      },
      &a);
  if (st == RDM_OK) {
    if (n_sub) *n_sub = n;
    if (nnz_sub) *nnz_sub = nnz;
  }
  return st;
}

rdm_status rdm_saint_wait(rdm_saint* s) {
  if (!s) return RDM_ERR_ARG;
  if (s->sst && s->iteration >= 0 && cudaStreamWaitEvent(s->ctx->stream, s->ev_done[s->cur], 0) != cudaSuccess)
    return RDM_ERR_CUDA;
  return RDM_OK;
}

rdm_status rdm_saint_subgraph(const rdm_saint* s, const int32_t** nodes, const int64_t** rowptr,
                              const int32_t** col, const float** val, int64_t* n, int64_t* nnz) {
  if (!s) return RDM_ERR_ARG;
  if (s->iteration < 0) return RDM_ERR_STATE;
  if (s->sst) cudaStreamSynchronize(s->sst);   // the build may still be finishing on the sampler stream
  const Csr& S = s->graph().A;
  if (nodes) *nodes = s->nodes_b[s->cur]->as<int32_t>();
  if (rowptr) *rowptr = S.rowptr->as<int64_t>();
  if (col) *col = S.col->as<int32_t>();
  if (val) *val = S.val->as<float>();
  if (n) *n = S.n;
  if (nnz) *nnz = S.nnz;
  return RDM_OK;
}

}  // extern "C"
