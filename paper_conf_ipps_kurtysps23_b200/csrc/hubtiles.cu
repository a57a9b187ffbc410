// hubtiles.cu — binary hub tiles: the dense part of the SpMM's adjacency on
// the kind::f16 tensor cores (sm_100a).
//
// PAPER.md §III-A (L102-104, Fig. 2a): the aggregation Out = A·In of a column
// slice needs no communication (A replicated).  This file changes HOW the
// product is computed for the part of A that is dense enough to be a genuine
// contraction, never WHAT is computed (A·X up to fp32 summation order, L323).
//
// Observation.  The GCN adjacency is Â = D̃^-1/2 (A+I) D̃^-1/2 (reading R6):
// every stored value factors as â_ij = s_i·s_j with s_i = deg_i^-1/2, i.e. Â is
// a row/column-scaled 0/1 matrix.  On the R-MAT graphs the highest-degree
// vertices form a block-dense region (profiles/r1_core_experiment.md: the
// mutual block of the top 4,096 vertices is 74 % non-zero), and rank-ordered
// 128 x 128 blocks down to a few % density still hold most entries.  So:
//
//   (Â X)_i = s_i · Σ_j b_ij · (s_j X_j)        b_ij ∈ {0, 1}
//
// * b is exact in bf16 → the A operand of a kind::f16 MMA is exact, and a
//   tile costs 32 KB (vs 64 KB fp32) of HBM;
// * X'_j = s_j X_j (fp32) is split into three bf16 pieces hi + mid + lo
//   (8 + 8 + 8 significant bits = fp32's 24), so b·X' = b·hi + b·mid + b·lo
//   with exact products and fp32 accumulation: fp32-class accuracy at 1.5x the
//   cost of one tf32 MMA (vs 3xTF32's 3 tf32 MMAs);
// * s_i is applied in the residual SpMM's epilogue, after the per-row-block
//   partial sums (fixed order: deterministic).
//
// The library verifies the factorisation at rdm_set_graph on every entry it
// moves into a tile (|â_ij − s_i s_j| ≤ 2^-21 â_ij; hypotheses deg^-1/2 and all
// ones).  Graphs whose values do not factor keep the fp32 dense hub core
// (spmm.cu build_core) or none.
//
// Kernel (persistent, one CTA per SM, warp-specialised like gemm_tc.cu):
//   warp 0 TMA producer: per 64-wide k stage the A tile half (128 x 64 bf16,
//          16 KB) and the three B pieces (n_mma x 64 bf16 each), 128B swizzle
//   warp 1 MMA issuer: 4 k16 steps x 3 pieces of tcgen05.mma kind::f16 per
//          stage into a double-buffered TMEM accumulator (128 x n_mma fp32)
//   warp 2 TMEM allocator
//   warps 4-7 epilogue: tcgen05.ld → partial rows of the work item → global
// A work item is a run of ≤ `chunk` tiles of one 128-row block; its 128 x w
// partial goes to part[item] and the SpMM epilogue sums the items of the row's
// block in item order.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "internal.h"
#include "tc_ptx.h"

namespace rdm {
namespace {
using namespace tc;

constexpr int TK = 128;                 // tile edge (rows and columns, rank space)
constexpr int SK = 64;                  // bf16 k per 128-byte swizzle row = per stage
constexpr int kMaxK2 = 262144;          // rank range considered (2048 row blocks)
constexpr int kSmemBudget = 220 * 1024;

// kind::f16 instruction descriptor: D f32, A/B bf16, K-major both, M = 128.
__host__ __device__ constexpr uint32_t idesc_bf16(int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

__global__ void __launch_bounds__(256, 1)
hub_tile_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB0,
                const __grid_constant__ CUtensorMap tmB1, const __grid_constant__ CUtensorMap tmB2,
                const int32_t* __restrict__ tile_cb, const int32_t* __restrict__ item_tb, int n_items,
                int tiles_n, int n_mma, int64_t w, float* __restrict__ part, int64_t ldp, int S,
                int stage_bytes) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint64_t* full = (uint64_t*)(smem + S * stage_bytes);
  uint64_t* empty = full + S;
  uint64_t* tfull = empty + S;   // [2]
  uint64_t* tempty = tfull + 2;  // [2]
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int total = n_items * tiles_n;
  const int bpiece = n_mma * 128;                 // bytes of one B piece per stage
  auto A_st = [&](int s) { return smem + s * stage_bytes; };
  auto B_st = [&](int s, int p) { return smem + s * stage_bytes + 16384 + p * bpiece; };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "n"(256));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      const uint32_t bytes = 16384 + 3 * bpiece;
      uint32_t kc = 0;
      for (int t = blockIdx.x; t < total; t += gridDim.x) {
        const int item = t / tiles_n;
        const int n0 = (t % tiles_n) * 128;
        const int tb = item_tb[item], te = item_tb[item + 1];
        for (int tile = tb; tile < te; ++tile) {
          const int kcol = tile_cb[tile] * TK;
          for (int h = 0; h < TK / SK; ++h, ++kc) {
            const int s = kc % S;
            if (kc >= (uint32_t)S) mbar_wait(&empty[s], ((kc / S) - 1) & 1);
            mbar_expect_tx(&full[s], bytes);
            tma_load_2d(A_st(s), &tmA, &full[s], h * SK, tile * TK);
            tma_load_2d(B_st(s, 0), &tmB0, &full[s], kcol + h * SK, n0);
            tma_load_2d(B_st(s, 1), &tmB1, &full[s], kcol + h * SK, n0);
            tma_load_2d(B_st(s, 2), &tmB2, &full[s], kcol + h * SK, n0);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      const uint32_t idesc = idesc_bf16(n_mma);
      uint32_t kc = 0;
      int it = 0;
      for (int t = blockIdx.x; t < total; t += gridDim.x, ++it) {
        const int item = t / tiles_n;
        const int nst = (item_tb[item + 1] - item_tb[item]) * (TK / SK);
        const int acc = it & 1;
        if (it >= 2) mbar_wait(&tempty[acc], ((it >> 1) - 1) & 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * 128;
        for (int st = 0; st < nst; ++st, ++kc) {
          const int s = kc % S;
          mbar_wait(&full[s], (kc / S) & 1);
          tc_fence_after();
          const uint32_t a = smem_u32(A_st(s));
          const uint32_t b0 = smem_u32(B_st(s, 0)), b1 = smem_u32(B_st(s, 1)), b2 = smem_u32(B_st(s, 2));
#pragma unroll
          for (int j = 0; j < SK / 16; ++j) {   // k16 steps: 32 bytes along the swizzled row
            const uint64_t da = sdesc(a + j * 32, 16, 1024);
            tc_mma_f16(d_tmem, da, sdesc(b0 + j * 32, 16, 1024), idesc, (st > 0 || j > 0) ? 1u : 0u);
            tc_mma_f16(d_tmem, da, sdesc(b1 + j * 32, 16, 1024), idesc, 1u);
            tc_mma_f16(d_tmem, da, sdesc(b2 + j * 32, 16, 1024), idesc, 1u);
          }
          tc_commit(&empty[s]);
        }
        tc_commit(&tfull[acc]);
      }
    }
  } else if (warp >= 4) {
    const int q = warp & 3;
    int it = 0;
    for (int t = blockIdx.x; t < total; t += gridDim.x, ++it) {
      const int item = t / tiles_n;
      const int64_t n0 = (int64_t)(t % tiles_n) * 128;
      const int acc = it & 1;
      mbar_wait_sleep(&tfull[acc], (it >> 1) & 1);
      tc_fence_after();
      float* prow = part + ((int64_t)item * TK + q * 32 + lane) * ldp + n0;
      for (int c0 = 0; c0 < n_mma; c0 += 32) {
        if (n0 + c0 >= w) break;
        uint32_t r[32];
        tmem_ld32(tmem_base + acc * 128 + ((uint32_t)(q * 32) << 16) + (uint32_t)c0, r);
#pragma unroll
        for (int i = 0; i < 32; i += 4)
          if (n0 + c0 + i < w)
            *reinterpret_cast<float4*>(prow + c0 + i) =
                make_float4(__uint_as_float(r[i]), __uint_as_float(r[i + 1]), __uint_as_float(r[i + 2]),
                            __uint_as_float(r[i + 3]));
      }
      tc_fence_before();
      mbar_arrive(&tempty[acc]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(256));
  }
}

// B pieces: P_p[n][k] = piece p of s_k · X[hub_k][n] (K-major rows of length K2),
// transposed through shared memory.  hi = bf16(x), mid = bf16(x − hi),
// lo = bf16(x − hi − mid); the differences are exact in fp32.
__global__ void tile_panels_kernel(const float* __restrict__ X, int64_t ldx, const int32_t* __restrict__ hub_ids,
                                   const float* __restrict__ scale, int64_t K2, int64_t w,
                                   __nv_bfloat16* __restrict__ p0, __nv_bfloat16* __restrict__ p1,
                                   __nv_bfloat16* __restrict__ p2) {
  __shared__ float t[64][33];
  const int64_t k0 = (int64_t)blockIdx.x * 64, n0 = (int64_t)blockIdx.y * 32;
  for (int i = threadIdx.y; i < 64; i += 8) {
    const int64_t k = k0 + i, n = n0 + threadIdx.x;
    t[i][threadIdx.x] = (n < w) ? __ldg(scale + k) * __ldg(X + (int64_t)__ldg(hub_ids + k) * ldx + n) : 0.f;
  }
  __syncthreads();
  for (int i = threadIdx.y; i < 32; i += 8) {
    const int64_t n = n0 + i;
    if (n >= w) break;
#pragma unroll
    for (int hk = 0; hk < 2; ++hk) {
      const int kk = hk * 32 + threadIdx.x;
      const float x = t[kk][i];
      const __nv_bfloat16 h = __float2bfloat16_rn(x);
      const float r1 = x - __bfloat162float(h);
      const __nv_bfloat16 m = __float2bfloat16_rn(r1);
      const __nv_bfloat16 l = __float2bfloat16_rn(r1 - __bfloat162float(m));
      const int64_t o = n * K2 + k0 + kk;
      p0[o] = h;
      p1[o] = m;
      p2[o] = l;
    }
  }
}

PFN_cuTensorMapEncodeTiled_v12000 encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    RDM_CUDA(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q));
    if (q != cudaDriverEntryPointSuccess || !p) throw Error(RDM_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
    fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
  }
  return fn;
}

// 2-D bf16 map: inner (contiguous) x outer, row stride ld elements, box
// {64, box_outer}, 128-byte swizzle, out-of-bounds rows read as zeros.
CUtensorMap bf16_map(const void* base, int64_t inner, int64_t outer, int64_t ld, int box_outer) {
  CUtensorMap m;
  cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)outer};
  cuuint64_t strides[1] = {(cuuint64_t)(ld * 2)};
  cuuint32_t box[2] = {(cuuint32_t)SK, (cuuint32_t)box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = encode()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(RDM_ERR_CUDA, "cuTensorMapEncodeTiled (bf16) failed (" + std::to_string((int)r) + ")");
  return m;
}

// Per-call cost model (B200, calibrated against profiles/r1_core_experiment.md
// and the hub-tile timings): a CSR entry costs ≈ 24 ps·(w/128)^0.55 (L2-gather
// bound), a tile ≈ ceil(w/128)·(4 + 6·min(w,128)/128) ns (A-tile stream +
// 3 bf16 MMAs), plus ≈ 20 µs of fixed per-call cost.
double csr_entry_s(int64_t w) { return 24e-12 * std::pow((double)w / 128.0, 0.55); }
double tile_s(int64_t w) {
  return (double)ceil_div(w, 128) * (4e-9 + 6e-9 * (double)std::min<int64_t>(w, 128) / 128.0);
}
}  // namespace

bool hub_tiles_pay(const Core& c, int64_t w) {
  if (!c.n_tiles) return false;
  if (c.forced) return true;
  return (double)c.nnz * csr_entry_s(w) > (double)c.n_tiles * tile_s(w) + 20e-6;
}

void hub_tiles_product(rdm_ctx* ctx, const Core& c, const float* X, int64_t ldx, int64_t w, float* part,
                       int64_t ldp) {
  const int64_t K2 = c.K2;
  __nv_bfloat16* pan = reinterpret_cast<__nv_bfloat16*>(ensure_ws(ctx->ws_core_b, (size_t)3 * w * K2 * 2));
  dim3 pg((unsigned)(K2 / 64), (unsigned)ceil_div(w, 32));
  tile_panels_kernel<<<pg, dim3(32, 8), 0, ctx->stream>>>(X, ldx, c.hub_ids->as<int32_t>(), c.scale->as<float>(), K2,
                                                        w, pan, pan + w * K2, pan + 2 * w * K2);
  RDM_LAUNCHED(ctx);
  const int n_mma = (int)std::min<int64_t>(128, ((w + 15) / 16) * 16);
  const int tiles_n = (int)ceil_div(w, 128);
  const CUtensorMap ta = bf16_map(c.tiles->ptr, TK, c.n_tiles * TK, TK, TK);
  const CUtensorMap b0 = bf16_map(pan, K2, w, K2, n_mma);
  const CUtensorMap b1 = bf16_map(pan + w * K2, K2, w, K2, n_mma);
  const CUtensorMap b2 = bf16_map(pan + 2 * w * K2, K2, w, K2, n_mma);
  const int stage_bytes = 16384 + 3 * n_mma * 128;
  const int S = std::min(8, (kSmemBudget - 1024 - 256) / stage_bytes);
  const int smem = S * stage_bytes + 1024 + 256;
  RDM_CUDA(cudaFuncSetAttribute(hub_tile_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  const int64_t total = c.n_items * tiles_n;
  const unsigned grid = (unsigned)std::min<int64_t>(total, ctx->num_sms);
  hub_tile_kernel<<<grid, 256, smem, ctx->stream>>>(ta, b0, b1, b2, c.tile_cb->as<int32_t>(), c.item_tb->as<int32_t>(),
                                                   (int)c.n_items, tiles_n, n_mma, w, part, ldp, S, stage_bytes);
  RDM_LAUNCHED(ctx);
}

// Host builder (one-time, rdm_set_graph, symmetric A).  Env (experiments and
// tests): RDM_NO_TILES=1 disables, RDM_TILE_MIN_NNZ=m selects every block with
// ≥ m entries and uses the tiles at every width, RDM_TILE_K2=k limits the rank range.
bool build_hub_tiles(rdm_ctx* ctx, Csr& A, const int64_t* rp, const int32_t* col, const float* val) {
  const char* off = getenv("RDM_NO_TILES");
  if (off && atoi(off)) return false;
  const int64_t n = A.n, nnz = A.nnz;
  if (n < TK || nnz == 0) return false;
  std::vector<int32_t> order(n);
  for (int64_t i = 0; i < n; ++i) order[i] = (int32_t)i;
  std::stable_sort(order.begin(), order.end(),
                   [&](int32_t a, int32_t b) { return rp[a + 1] - rp[a] > rp[b + 1] - rp[b]; });
  std::vector<int32_t> rank(n);
  for (int64_t i = 0; i < n; ++i) rank[order[i]] = (int32_t)i;
  int64_t K2 = std::min<int64_t>(n / TK * TK, kMaxK2);
  if (const char* e = getenv("RDM_TILE_K2")) K2 = std::min<int64_t>(K2, std::max<int64_t>(TK, atoll(e) / TK * TK));
  const int64_t nrb = K2 / TK;
  // entries per rank block
  std::vector<int32_t> cnt((size_t)nrb * nrb, 0);
  for (int64_t i = 0; i < n; ++i) {
    const int64_t ri = rank[i];
    if (ri >= K2) continue;
    for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
      const int64_t rj = rank[col[j]];
      if (rj < K2) cnt[(size_t)(ri / TK) * nrb + rj / TK]++;
    }
  }
  bool forced = false;
  int64_t min_nnz = (int64_t)std::ceil(tile_s(128) / csr_entry_s(128));
  if (const char* e = getenv("RDM_TILE_MIN_NNZ")) {
    min_nnz = std::max<int64_t>(1, atoll(e));
    forced = true;
  }
  std::vector<int32_t> tile_id((size_t)nrb * nrb, -1);
  std::vector<int32_t> tile_cb;
  std::vector<int32_t> rb_first(nrb + 1, 0);
  int64_t moved = 0, max_blk = 0;
  for (int64_t rb = 0; rb < nrb; ++rb) {
    rb_first[rb] = (int32_t)tile_cb.size();
    for (int64_t cb = 0; cb < nrb; ++cb) {
      const int32_t c = cnt[(size_t)rb * nrb + cb];
      if (c >= min_nnz) {
        tile_id[(size_t)rb * nrb + cb] = (int32_t)tile_cb.size();
        tile_cb.push_back((int32_t)cb);
        moved += c;
        max_blk = std::max(max_blk, std::max(rb, cb));
      }
    }
  }
  rb_first[nrb] = (int32_t)tile_cb.size();
  const int64_t n_tiles = (int64_t)tile_cb.size();
  if (n_tiles == 0 || n_tiles > (int64_t)INT32_MAX / (TK * TK)) return false;
  if (!forced && (double)moved * csr_entry_s(128) < (double)n_tiles * tile_s(128) + 100e-6) return false;
  // factorisation â_ij = s_i s_j on every moved entry: s = deg^-1/2 (GCN), else s = 1
  std::vector<double> s(n);
  bool ok = false;
  for (int hyp = 0; hyp < 2 && !ok; ++hyp) {
    for (int64_t i = 0; i < n; ++i) s[i] = hyp == 0 ? 1.0 / std::sqrt((double)(rp[i + 1] - rp[i])) : 1.0;
    ok = true;
    for (int64_t i = 0; i < n && ok; ++i) {
      const int64_t ri = rank[i];
      if (ri >= K2) continue;
      for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
        const int64_t rj = rank[col[j]];
        if (rj >= K2 || tile_id[(size_t)(ri / TK) * nrb + rj / TK] < 0) continue;
        const double f = s[i] * s[col[j]];
        if (!(std::fabs((double)val[j] - f) <= std::ldexp(f, -21))) {
          ok = false;
          break;
        }
      }
    }
  }
  if (!ok) return false;
  Core& c = A.core;
  c.forced = forced;
  c.K2 = (max_blk + 1) * TK;
  c.n_rb = c.K2 / TK;
  c.n_tiles = n_tiles;
  c.nnz = moved;
  // work items: runs of ≤ chunk tiles of one row block (≈ 4 items per SM)
  const int64_t chunk = std::max<int64_t>(4, ceil_div(n_tiles, (int64_t)ctx->num_sms * 4));
  std::vector<int32_t> item_tb, rb_item(c.n_rb + 1, 0);
  for (int64_t rb = 0; rb < c.n_rb; ++rb) {
    rb_item[rb] = (int32_t)item_tb.size();
    const int64_t t0 = rb_first[rb], T = rb_first[rb + 1] - t0;
    const int64_t nit = ceil_div(T, chunk);
    for (int64_t k = 0; k < nit; ++k) item_tb.push_back((int32_t)(t0 + T * k / nit));
  }
  rb_item[c.n_rb] = (int32_t)item_tb.size();
  c.n_items = (int64_t)item_tb.size();
  item_tb.push_back((int32_t)n_tiles);
  // tiles (bf16 0/1, filled one row block at a time) and the residual CSR
  c.tiles.reset(new DevBuf((size_t)n_tiles * TK * TK * 2));
  std::vector<int64_t> rrp(n + 1, 0);
  auto in_tile = [&](int64_t ri, int64_t rj) {
    return ri < K2 && rj < K2 && tile_id[(size_t)(ri / TK) * nrb + rj / TK] >= 0;
  };
  std::vector<uint16_t> buf;
  for (int64_t rb = 0; rb < c.n_rb; ++rb) {
    const int64_t t0 = rb_first[rb], T = rb_first[rb + 1] - t0;
    if (!T) continue;
    buf.assign((size_t)T * TK * TK, 0);
    for (int64_t r = 0; r < TK; ++r) {
      const int64_t v = order[rb * TK + r];
      for (int64_t j = rp[v]; j < rp[v + 1]; ++j) {
        const int64_t rj = rank[col[j]];
        if (!in_tile(rb * TK + r, rj)) continue;
        const int64_t t = tile_id[(size_t)rb * nrb + rj / TK] - t0;
        uint16_t& e = buf[(size_t)t * TK * TK + r * TK + (rj % TK)];
        float f = 0.f;
        if (e) {
          uint32_t u = (uint32_t)e << 16;
          std::memcpy(&f, &u, 4);
        }
        f += 1.f;   // duplicate entries add up (small integers are exact in bf16)
        uint32_t u;
        std::memcpy(&u, &f, 4);
        e = (uint16_t)(u >> 16);
      }
    }
    RDM_CUDA(cudaMemcpy(c.tiles->as<uint8_t>() + (size_t)t0 * TK * TK * 2, buf.data(), buf.size() * 2,
                        cudaMemcpyHostToDevice));
  }
  for (int64_t i = 0; i < n; ++i) {
    int64_t keep = 0;
    for (int64_t j = rp[i]; j < rp[i + 1]; ++j) keep += !in_tile(rank[i], rank[col[j]]);
    rrp[i + 1] = rrp[i] + keep;
  }
  const int64_t rnnz = rrp[n];
  std::vector<int32_t> rcol(std::max<int64_t>(rnnz, 1));
  std::vector<float> rval(std::max<int64_t>(rnnz, 1));
  for (int64_t i = 0; i < n; ++i) {
    int64_t o = rrp[i];
    for (int64_t j = rp[i]; j < rp[i + 1]; ++j)
      if (!in_tile(rank[i], rank[col[j]])) {
        rcol[o] = col[j];
        rval[o] = val[j];
        ++o;
      }
  }
  std::vector<float> sc(c.K2);
  for (int64_t k = 0; k < c.K2; ++k) sc[k] = (float)s[order[k]];
  std::vector<int32_t> slot(n);
  for (int64_t v = 0; v < n; ++v) slot[v] = rank[v] < c.K2 ? rank[v] : -1;
  auto up = [&](std::unique_ptr<DevBuf>& b, const void* p, size_t bytes) {
    b.reset(new DevBuf(std::max<size_t>(bytes, 16)));
    if (bytes) RDM_CUDA(cudaMemcpy(b->ptr, p, bytes, cudaMemcpyHostToDevice));
  };
  up(c.tile_cb, tile_cb.data(), n_tiles * 4);
  up(c.item_tb, item_tb.data(), item_tb.size() * 4);
  up(c.rb_item, rb_item.data(), rb_item.size() * 4);
  up(c.scale, sc.data(), sc.size() * 4);
  up(c.hub_ids, order.data(), c.K2 * 4);
  up(c.hub_slot, slot.data(), n * 4);
  c.resid.reset(new Csr());
  Csr& R = *c.resid;
  R.n = n;
  R.nnz = rnnz;
  up(R.rowptr, rrp.data(), (n + 1) * 8);
  up(R.col, rcol.data(), rnnz * 4);
  up(R.val, rval.data(), rnnz * 4);
  build_bins(ctx, R, rrp.data());
  return true;
}

}  // namespace rdm
