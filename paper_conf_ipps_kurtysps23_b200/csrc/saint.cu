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
// then the host builds the row bins from rowptr_s (one D2H copy).
#include <cub/cub.cuh>

#include <cmath>

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

// Induced-subgraph extraction is entry-parallel: each sampled row's ORIGINAL
// adjacency list (random walks favour hubs: rows of 10^4-10^5 entries) is cut
// into kSeg-entry segments, one warp per segment, so a hub row does not
// serialise on one warp.
constexpr int kSeg = 1024;

// nseg[i] = segments of sampled row i (0 for i >= n_sub)
__global__ void rowseg_kernel(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ nodes,
                              int64_t n_cap, const unsigned long long* scal, int32_t* __restrict__ nseg) {
  const int64_t n = (int64_t)scal[0];
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i <= n_cap;
       i += (int64_t)gridDim.x * blockDim.x) {
    int32_t c = 0;
    if (i < n) {
      const int32_t v = nodes[i];
      c = (int32_t)((rowptr[v + 1] - rowptr[v] + kSeg - 1) / kSeg);
    }
    nseg[i] = c;
  }
}

__global__ void segrow_kernel(const int32_t* __restrict__ nseg, const int32_t* __restrict__ segoff,
                              const unsigned long long* scal, int32_t* __restrict__ seg_row) {
  const int64_t n = (int64_t)scal[0];
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    for (int32_t k = 0; k < nseg[i]; ++k) seg_row[segoff[i] + k] = (int32_t)i;
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
    const int32_t i = seg_row[sg];
    const int32_t v = nodes[i];
    const int64_t e = rowptr[v + 1];
    const int64_t b = rowptr[v] + (sg - segoff[i]) * kSeg;
    const int64_t end = b + kSeg < e ? b + kSeg : e;
    int c = 0;
    for (int64_t k = b + lane; k < end; k += 32) c += flag[__ldg(col + k)] ? 1 : 0;
#pragma unroll
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if (lane == 0) {
      cnt[sg] = c;
      if (c) {
        atomicAdd(deg + i, (unsigned long long)c);
        atomicAdd(scal + 1, (unsigned long long)c);
      }
    }
  }
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
    const int32_t i = seg_row[sg];
    const int32_t v = nodes[i];
    const int64_t e = rowptr[v + 1];
    const int64_t b = rowptr[v] + (sg - segoff[i]) * kSeg;
    const int64_t end = b + kSeg < e ? b + kSeg : e;
    int64_t at0 = pos[sg];
    const double di = (double)deg[i];
    for (int64_t k0 = b; k0 < end; k0 += 32) {
      const int64_t k = k0 + lane;
      const int32_t u = k < end ? __ldg(col + k) : 0;
      const bool keep = k < end && flag[u];
      const unsigned m = __ballot_sync(0xffffffffu, keep);
      if (keep) {
        const int64_t at = at0 + __popc(m & ((1u << lane) - 1u));
        const int32_t j = map[u];
        col_s[at] = j;
        val_s[at] = (float)(1.0 / sqrt(di * (double)deg[j]));
      }
      at0 += __popc(m);
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

void sample(rdm_saint* s, int64_t it, int64_t* n_out, int64_t* nnz_out) {
  rdm_ctx* ctx = s->ctx;
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
  int32_t* nodes = reinterpret_cast<int32_t*>(ensure_ws(s->nodes, cap * sizeof(int32_t)));
  unsigned long long* deg = reinterpret_cast<unsigned long long*>(ensure_ws(s->deg, (cap + 1) * 8));
  // segment tables: nseg[cap+1] | segoff[cap+1] | seg_row[seg_cap] (int32); cnt | pos (int64)
  int32_t* nseg = reinterpret_cast<int32_t*>(ensure_ws(s->seg, (2 * (cap + 1) + seg_cap) * 4 + 16));
  int32_t* segoff = nseg + (cap + 1);
  int32_t* seg_row = segoff + (cap + 1);
  int64_t* cnt = reinterpret_cast<int64_t*>(ensure_ws(s->rps, 2 * seg_cap * sizeof(int64_t)));
  int64_t* pos = cnt + seg_cap;
  unsigned long long* scal = reinterpret_cast<unsigned long long*>(ensure_ws(s->scal, 64));
  size_t tb[4] = {0, 0, 0, 0};
  RDM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb[0], flag, map, (int)N, ctx->stream));
  RDM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb[1], nseg, segoff, (int)(cap + 1), ctx->stream));
  RDM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb[2], cnt, pos, (int)seg_cap, ctx->stream));
  int64_t* rp_dummy = nullptr;
  RDM_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb[3], deg, rp_dummy, (int)(cap + 1), ctx->stream));
  const size_t tbm = std::max(std::max(tb[0], tb[1]), std::max(tb[2], tb[3]));
  void* tmp = ensure_ws(s->tmp, tbm);
  auto scan = [&](auto* in, auto* out, int64_t count) {
    size_t t = tbm;
    RDM_CUDA(cub::DeviceScan::ExclusiveSum(tmp, t, in, out, (int)count, ctx->stream));
  };

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
  scan(flag, map, N);
  compact_kernel<<<grid_of(ctx, N, 256), 256, 0, ctx->stream>>>(flag, map, N, nodes, scal);
  RDM_LAUNCHED(ctx);
  rowseg_kernel<<<grid_of(ctx, cap + 1, 256), 256, 0, ctx->stream>>>(A.rowptr->as<int64_t>(), nodes,
                                                                       cap, scal, nseg);
  RDM_LAUNCHED(ctx);
  scan(nseg, segoff, cap + 1);
  segrow_kernel<<<grid_of(ctx, cap, 256), 256, 0, ctx->stream>>>(nseg, segoff, scal, seg_row);
  RDM_LAUNCHED(ctx);
  count_kernel<<<grid_of(ctx, seg_cap * 32, 256), 256, 0, ctx->stream>>>(
      A.rowptr->as<int64_t>(), A.col->as<int32_t>(), flag, nodes, seg_row, segoff, cap, cnt, deg, scal);
  RDM_LAUNCHED(ctx);
  unsigned long long hs[2];
  RDM_CUDA(cudaMemcpyAsync(hs, scal, sizeof(hs), cudaMemcpyDeviceToHost, ctx->stream));
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  const int64_t n = (int64_t)hs[0], nnz = (int64_t)hs[1];
  if (n > cap) throw Error(RDM_ERR_STATE, "saint: subgraph larger than its capacity");

  Graph& G = s->graph;
  Csr& S = G.A;
  int64_t* rp = reinterpret_cast<int64_t*>(ensure_ws(S.rowptr, (cap + 1) * sizeof(int64_t)));
  int32_t* cs = reinterpret_cast<int32_t*>(ensure_ws(S.col, std::max<int64_t>(nnz, 1) * sizeof(int32_t)));
  float* vs = ensure_ws(S.val, std::max<int64_t>(nnz, 1) * sizeof(float));
  // rowptr_s: prefix of d (zero beyond n); segment output offsets: prefix of c
  scan(deg, rp, cap + 1);
  scan(cnt, pos, seg_cap);
  fill_kernel<<<grid_of(ctx, seg_cap * 32, 256), 256, 0, ctx->stream>>>(
      A.rowptr->as<int64_t>(), A.col->as<int32_t>(), flag, map, nodes, seg_row, segoff, cap, deg, pos,
      cs, vs);
  RDM_LAUNCHED(ctx);
  std::vector<int64_t> rph(n + 1);
  RDM_CUDA(cudaMemcpyAsync(rph.data(), rp, (n + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, ctx->stream));
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  S.n = n;
  S.nnz = nnz;
  build_bins(ctx, S, rph.data());
  G.n = n;
  G.nnz = nnz;
  G.symmetric = true;
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
  delete s;
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

rdm_status rdm_saint_subgraph(const rdm_saint* s, const int32_t** nodes, const int64_t** rowptr,
                              const int32_t** col, const float** val, int64_t* n, int64_t* nnz) {
  if (!s) return RDM_ERR_ARG;
  if (s->iteration < 0) return RDM_ERR_STATE;
  const Csr& S = s->graph.A;
  if (nodes) *nodes = s->nodes->as<int32_t>();
  if (rowptr) *rowptr = S.rowptr->as<int64_t>();
  if (col) *col = S.col->as<int32_t>();
  if (val) *val = S.val->as<float>();
  if (n) *n = S.n;
  if (nnz) *nnz = S.nnz;
  return RDM_OK;
}

}  // extern "C"
