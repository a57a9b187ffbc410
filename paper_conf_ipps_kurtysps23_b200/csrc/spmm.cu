// spmm.cu — communication-free CSR SpMM on a feature-column slice (sm_100a).
//
// PAPER.md §III-A (L102-104, Fig. 2a): Out = M·In needs no communication when
// M (here the adjacency A) is replicated and In/Out are column ("vertically")
// sliced.  The GCN aggregation of eq. (1) is Aᵀ·H (L69-71) and the backward
// products of eq. (3)(4) are A·G (L77-79).  Each GPU multiplies the WHOLE
// replicated CSR by its N x w column slice.
//
// Design (B200):
//  * Work items are (light row) or (fixed-size nnz segment of a heavy row).
//    Light rows (deg <= kSeg) are processed warp-per-row in descending-degree
//    order (LPT), heavy rows are cut into kSeg-nnz segments processed
//    warp-per-segment, whose partial rows are summed in segment order by a
//    second tiny kernel: deterministic, no float atomics (the "CTA per heavy
//    row" variant generalised to any degree).
//  * Inside a warp, G lanes cover one nnz × (4G) columns with 128-bit gathers
//    of the H row; 32/G nnz are in flight per warp step, so narrow slices
//    (w = 16 at P = 8) still issue full-warp gathers.  Columns beyond 128 are
//    handled by blockIdx.y chunks.
//  * CSR col/val are streamed with evict-first loads (__ldcs) so the gathered
//    H slice keeps L2; gathers use the read-only path (__ldg).
//  * Fused epilogue: bias, ReLU, Hadamard mask 1[mask > 0] (eq. 3's σ').
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <vector>

#include <cuda_bf16.h>
#include <cub/cub.cuh>

#include "internal.h"

// load form of the gathered input rows (timing experiments may rebuild with
// another cache operator, tools/build_variant.sh)
#ifndef RDM_GATHER_LD
#define RDM_GATHER_LD __ldg
#endif

namespace rdm {
namespace {

constexpr int kWarps = 8;            // warps per CTA
constexpr int64_t kSeg = 2048;       // nnz per heavy-row segment / light-row cap
constexpr unsigned kFull = 0xffffffffu;

struct Epi {
  int flags;
  const float* bias;
  const float* mask;
  int64_t ld_mask;
  int64_t w;
  const float* core;        // hub-core product (K x ld_core) or null
  int64_t ld_core;
  const int32_t* hub_slot;  // int32[N], -1 for non-hubs
  const float* tpart;       // binary hub tiles: per-item partials (n_items x 2^item_shift x ld_tpart) or null
  int64_t ld_tpart;
  const int32_t* rb_item;   // item range of each block of 2^item_shift ranks
  int item_shift;           // 7: items of one row block; 8: of a row-block pair
  const float* tscale;      // row scale r_i of hub slot i (a_ij = r_i c_j)
  Scatter scat;             // fused col→row redistribution (scat.P == 0: off)
  const float* rscale;      // factored bf16 path: s_i per row (applied first), or null
};

// Fused col→row redistribution: row r of my column slice (columns c..c+3 of
// it) goes to the row-slice buffer of r's owner, at my global column offset.
__device__ __forceinline__ void scatter_row_store(const Scatter& s, int64_t r, int64_t c, float4 v) {
  if (c >= s.my_w) return;  // slice padding is not part of the row layout
  int q = 0;
  while (q + 1 < s.P && s.lo[q + 1] <= r) ++q;
  float* d = s.ptr[q] + (r - s.lo[q]) * s.ld[q] + s.my_off + c;
  if (c + 4 <= s.my_w) {
    *reinterpret_cast<float4*>(d) = v;
  } else {
    d[0] = v.x;
    if (c + 1 < s.my_w) d[1] = v.y;
    if (c + 2 < s.my_w) d[2] = v.z;
  }
}

__device__ __forceinline__ float4 apply_epi(float4 a, const Epi& e, int64_t row, int64_t c) {
  if (e.rscale) {   // factored rows: Σ_j bf16(s_j X_j) · s_i
    const float sc = __ldg(e.rscale + row);
    a.x *= sc; a.y *= sc; a.z *= sc; a.w *= sc;
  }
  if (e.core) {  // add the dense hub-core contribution of this row (fixed order: after the CSR sum)
    const int s = __ldg(e.hub_slot + row);
    if (s >= 0) {
      const float4 k = __ldg(reinterpret_cast<const float4*>(e.core + (int64_t)s * e.ld_core + c));
      a.x += k.x; a.y += k.y; a.z += k.z; a.w += k.w;
    }
  }
  if (e.tpart) {  // binary hub tiles: s_i · Σ_items partial (item order; after the CSR sum)
    const int s = __ldg(e.hub_slot + row);
    if (s >= 0) {
      const int blk = s >> e.item_shift, rr = s & ((1 << e.item_shift) - 1);
      const int i0 = __ldg(e.rb_item + blk), i1 = __ldg(e.rb_item + blk + 1);
      float4 t = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int it = i0; it < i1; ++it) {
        const float4 k = __ldg(reinterpret_cast<const float4*>(
            e.tpart + (((int64_t)it << e.item_shift) + rr) * e.ld_tpart + c));
        t.x += k.x; t.y += k.y; t.z += k.z; t.w += k.w;
      }
      const float sc = __ldg(e.tscale + s);
      a.x = fmaf(sc, t.x, a.x); a.y = fmaf(sc, t.y, a.y); a.z = fmaf(sc, t.z, a.z); a.w = fmaf(sc, t.w, a.w);
    }
  }
  if (e.flags & RDM_EPI_BIAS) {
    if (c + 0 < e.w) a.x += e.bias[c + 0];
    if (c + 1 < e.w) a.y += e.bias[c + 1];
    if (c + 2 < e.w) a.z += e.bias[c + 2];
    if (c + 3 < e.w) a.w += e.bias[c + 3];
  }
  if (e.flags & RDM_EPI_RELU) {
    a.x = fmaxf(a.x, 0.f); a.y = fmaxf(a.y, 0.f); a.z = fmaxf(a.z, 0.f); a.w = fmaxf(a.w, 0.f);
  }
  if (e.flags & RDM_EPI_MASK) {
    const float4 m = __ldg(reinterpret_cast<const float4*>(e.mask + row * e.ld_mask + c));
    a.x = m.x > 0.f ? a.x : 0.f;
    a.y = m.y > 0.f ? a.y : 0.f;
    a.z = m.z > 0.f ? a.z : 0.f;
    a.w = m.w > 0.f ? a.w : 0.f;
  }
  return a;
}

// Column-relabelled SpMM of DRAM-resident slices (see rank_panel): the input
// slice is gathered into rank order X'[r] = X[order[r]] (vertices ranked by
// how often the CSR references them) and the kernel streams a column array of
// ranks, so the hottest rows are contiguous (full 128-byte lines, one L2-sized
// prefix).  hw == 0: off (plain column ids into X).
struct Hot {
  const float* xh;        // N x ldh, rank order
  int64_t ldh;
  int hw;
};

// Warp computes Σ_{j in [beg,end)} val[j] · X[col[j], chunk columns].  A group
// of G lanes owns one nnz at a time; lane `sub` of the group loads float4
// chunks sub, sub+G, …, sub+(V-1)G of the row chunk (each warp-level load is a
// contiguous 16·G-byte run per group), so 32/G nnz are in flight per step and
// every lane issues V independent 128-bit gathers per nnz.  (col, val) of 32
// nnz are loaded once per batch, coalesced, and broadcast with shuffles (none
// when G = 1).  Result: lanes of group 0 hold the row-chunk sum.
template <int G, int V, int U>
__device__ __forceinline__ void warp_nnz_range(const int32_t* __restrict__ col,
                                               const float* __restrict__ val,
                                               const float* __restrict__ xb, int64_t ldx,
                                               int64_t beg, int64_t end, int lane, int c4n,
                                               float4 (&acc)[V]) {
  constexpr int NG = 32 / G;
  static_assert(G % U == 0, "U must divide G");
  const int g = lane / G, sub = lane % G;
#pragma unroll
  for (int v = 0; v < V; ++v) acc[v] = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t base = beg; base < end; base += 32) {
    const int64_t j = base + lane;
    int c = 0;
    float a = 0.f;
    if (j < end) {
      c = __ldcs(col + j);
      a = __ldcs(val + j);
    }
    const int cnt = (end - base) < 32 ? (int)(end - base) : 32;
    // U nnz per group are gathered before any of them is consumed (U·V
    // independent 128-bit loads in flight per lane); an nnz past the row's end
    // loads nothing and contributes 0·0.
    if constexpr (U == 1) {
      // one nnz per group at a time, skipped past the row's end
#pragma unroll
      for (int t = 0; t < G; ++t) {
        const int k = t * NG + g;
        const int cc = (G == 1) ? c : __shfl_sync(kFull, c, k);
        const float vv = (G == 1) ? a : __shfl_sync(kFull, a, k);
        if (k < cnt) {
          const float4* xr = reinterpret_cast<const float4*>(xb + (int64_t)cc * ldx);
          float4 x[V];
#pragma unroll
          for (int v = 0; v < V; ++v)
            if (v * G + sub < c4n) x[v] = RDM_GATHER_LD(xr + v * G + sub);
#pragma unroll
          for (int v = 0; v < V; ++v) {
            if (v * G + sub < c4n) {
              acc[v].x = fmaf(vv, x[v].x, acc[v].x);
              acc[v].y = fmaf(vv, x[v].y, acc[v].y);
              acc[v].z = fmaf(vv, x[v].z, acc[v].z);
              acc[v].w = fmaf(vv, x[v].w, acc[v].w);
            }
          }
        }
      }
    } else {
#pragma unroll
    for (int t0 = 0; t0 < G; t0 += U) {
      if (t0 * NG >= cnt) break;   // warp-uniform: the rest of the batch is past the row's end
      float4 x[U][V];
      float vv[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int k = (t0 + u) * NG + g;
        const int cc = (G == 1) ? c : __shfl_sync(kFull, c, k);
        vv[u] = (G == 1) ? a : __shfl_sync(kFull, a, k);
        const float4* xr = reinterpret_cast<const float4*>(xb + (int64_t)cc * ldx);
#pragma unroll
        for (int v = 0; v < V; ++v)
          x[u][v] = (k < cnt && v * G + sub < c4n) ? RDM_GATHER_LD(xr + v * G + sub) : make_float4(0.f, 0.f, 0.f, 0.f);
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          acc[v].x = fmaf(vv[u], x[u][v].x, acc[v].x);
          acc[v].y = fmaf(vv[u], x[u][v].y, acc[v].y);
          acc[v].z = fmaf(vv[u], x[u][v].z, acc[v].z);
          acc[v].w = fmaf(vv[u], x[u][v].w, acc[v].w);
        }
    }
    }
  }
#pragma unroll
  for (int off = G; off < 32; off <<= 1) {
#pragma unroll
    for (int v = 0; v < V; ++v) {
      acc[v].x += __shfl_xor_sync(kFull, acc[v].x, off);
      acc[v].y += __shfl_xor_sync(kFull, acc[v].y, off);
      acc[v].z += __shfl_xor_sync(kFull, acc[v].z, off);
      acc[v].w += __shfl_xor_sync(kFull, acc[v].w, off);
    }
  }
}

// One warp per work item: items [0, n_seg) are heavy-row segments (partial
// rows to `part`), items [n_seg, n_seg + n_light) are light rows (to out).
// blockIdx.y selects a 128-column chunk of the slice.
// Resident CTAs per SM: the gathers are latency-bound, so occupancy is capped
// by registers only as far as the V accumulators need (measured on the
// Reddit-shaped residual CSR: V = 4 best at 4 CTAs, V = 3 at 5, V ≤ 2 at 6).
// With U nnz in flight per group the load registers grow by U·V: occupancy
// by float4-sized register slots (accumulators + loads), s = V + U·V here.
constexpr int spmm_minb_slots(int s) { return s <= 4 ? 6 : s <= 6 ? 5 : s <= 8 ? 4 : s <= 12 ? 3 : 2; }
constexpr int spmm_minb(int V, int U) { return U == 1 ? (V >= 4 ? 4 : V == 3 ? 5 : 6) : spmm_minb_slots(V + U * V); }
template <int G, int V, int U>
__global__ void __launch_bounds__(kWarps * 32, spmm_minb(V, U))
spmm_kernel(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
            const float* __restrict__ val, const int32_t* __restrict__ light_rows,
            const int64_t* __restrict__ seg_start, const int32_t* __restrict__ seg_row,
            int64_t n_light, int64_t n_seg, const float* __restrict__ X, int64_t ldx,
            float* __restrict__ out, int64_t ld_out, float* __restrict__ part, int64_t ld_part,
            int64_t w4, int chunk4, Epi epi) {
  const int lane = threadIdx.x & 31;
  const int64_t item = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5);
  if (item >= n_seg + n_light) return;
  const int64_t cbase = (int64_t)blockIdx.y * chunk4 * 4;      // first column of the chunk
  const int64_t rem4 = (w4 - cbase) / 4;
  const int c4n = rem4 < chunk4 ? (int)rem4 : chunk4;          // float4 chunks in this chunk
  const int sub = lane % G;
  float4 acc[V];
  int32_t r;
  if (item < n_seg) {
    r = seg_row[item];
    const int64_t beg = seg_start[item];
    const int64_t end = min(beg + kSeg, rowptr[r + 1]);
    warp_nnz_range<G, V, U>(col, val, X + cbase, ldx, beg, end, lane, c4n, acc);
    if (lane < G) {
      float* dst = part + item * ld_part + cbase;
#pragma unroll
      for (int v = 0; v < V; ++v)
        if (v * G + sub < c4n) reinterpret_cast<float4*>(dst)[v * G + sub] = acc[v];
    }
  } else {
    r = light_rows[item - n_seg];
    warp_nnz_range<G, V, U>(col, val, X + cbase, ldx, rowptr[r], rowptr[r + 1], lane, c4n, acc);
    if (lane < G) {
      float* dst = out + (int64_t)r * ld_out + cbase;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const int ch = v * G + sub;
        if (ch < c4n) {
          const float4 o = apply_epi(acc[v], epi, r, cbase + 4 * ch);
          reinterpret_cast<float4*>(dst)[ch] = o;
          if (epi.scat.P) scatter_row_store(epi.scat, r, cbase + 4 * ch, o);
        }
      }
    }
  }
}

// Short light rows (degree <= the short threshold, the suffix of the
// descending-degree light-row list): a group of G lanes per ROW, 32/G rows
// per warp, U entries of its row in flight per group — short rows leave most
// of a warp-per-row idle and serialise the rowptr → col → gather chain
// (papers100M-shaped: average degree 15).  Same epilogue and stores.
template <int G, int V, int U, int NB = 32>
__global__ void __launch_bounds__(kWarps * 32)
spmm_short_kernel(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                  const float* __restrict__ val, const int32_t* __restrict__ rows, int64_t n_rows,
                  const float* __restrict__ X, int64_t ldx, float* __restrict__ out, int64_t ld_out,
                  int64_t w4, int chunk4, Epi epi) {
  constexpr int R = 32 / G;
  const int lane = threadIdx.x & 31;
  const int g = lane / G, sub = lane % G;
  const int64_t idx = ((int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5)) * R + g;
  const int64_t cbase = (int64_t)blockIdx.y * chunk4 * 4;
  const int64_t rem4 = (w4 - cbase) / 4;
  const int c4n = rem4 < chunk4 ? (int)rem4 : chunk4;
  const bool live = idx < n_rows;
  const int32_t r = live ? rows[idx] : 0;
  const int64_t beg = live ? rowptr[r] : 0, end = live ? rowptr[r + 1] : 0;
  const float* xb = X + cbase;
  float4 acc[V];
#pragma unroll
  for (int v = 0; v < V; ++v) acc[v] = make_float4(0.f, 0.f, 0.f, 0.f);
  // The row's first NB (col, val) in one coalesced load up front (NB/G per
  // lane of the group), handed out by shuffles: the loop below then exposes
  // one gather latency per step instead of a (col, val) load followed by the
  // gather.  Same entry order, same sums.
  constexpr int SL = NB / G;
  int pc[SL];
  float pv[SL];
#pragma unroll
  for (int s = 0; s < SL; ++s) {
    const int64_t j = beg + s * G + sub;
    const bool ok = j < end;
    pc[s] = ok ? __ldcs(col + j) : 0;
    pv[s] = ok ? __ldcs(val + j) : 0.f;
  }
  const int deg = (int)(end - beg);
  const int dmax = __reduce_max_sync(kFull, deg < NB ? deg : NB);
#pragma unroll
  for (int e0 = 0; e0 < NB; e0 += U) {
    if (e0 >= dmax) break;   // warp-uniform
    int c[U];
    float a[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = e0 + u;
      c[u] = __shfl_sync(kFull, pc[e / G], g * G + (e % G));
      a[u] = __shfl_sync(kFull, pv[e / G], g * G + (e % G));
    }
    float4 x[U][V];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v)
        x[u][v] = (e0 + u < deg && v * G + sub < c4n)
                      ? RDM_GATHER_LD(reinterpret_cast<const float4*>(xb + (int64_t)c[u] * ldx) + v * G + sub)
                      : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v) {
        acc[v].x = fmaf(a[u], x[u][v].x, acc[v].x);
        acc[v].y = fmaf(a[u], x[u][v].y, acc[v].y);
        acc[v].z = fmaf(a[u], x[u][v].z, acc[v].z);
        acc[v].w = fmaf(a[u], x[u][v].w, acc[v].w);
      }
  }
  // rows longer than NB (RDM_SPMM_SHORT > 64, experiments): the rest entry by entry
  for (int64_t j = beg + NB; j < end; j += U) {
    int c[U];
    float a[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const bool ok = j + u < end;
      c[u] = ok ? __ldcs(col + j + u) : 0;
      a[u] = ok ? __ldcs(val + j + u) : 0.f;
    }
    float4 x[U][V];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v)
        x[u][v] = (j + u < end && v * G + sub < c4n)
                      ? RDM_GATHER_LD(reinterpret_cast<const float4*>(xb + (int64_t)c[u] * ldx) + v * G + sub)
                      : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v) {
        acc[v].x = fmaf(a[u], x[u][v].x, acc[v].x);
        acc[v].y = fmaf(a[u], x[u][v].y, acc[v].y);
        acc[v].z = fmaf(a[u], x[u][v].z, acc[v].z);
        acc[v].w = fmaf(a[u], x[u][v].w, acc[v].w);
      }
  }
  if (!live) return;
  float* dst = out + (int64_t)r * ld_out + cbase;
#pragma unroll
  for (int v = 0; v < V; ++v) {
    const int ch = v * G + sub;
    if (ch < c4n) {
      const float4 o = apply_epi(acc[v], epi, r, cbase + 4 * ch);
      reinterpret_cast<float4*>(dst)[ch] = o;
      if (epi.scat.P) scatter_row_store(epi.scat, r, cbase + 4 * ch, o);
    }
  }
}

// RDM_PREC_FAST: the same walk over a bf16 copy of the slice.  A lane's
// 128-bit gather now carries 8 columns; bf16 → fp32 is exact (a shift), the
// products and sums stay fp32.  acc[v][0..1] = columns 8·ch + 0..3, + 4..7.
// fp32 += bf16 (low or high half of u) · 1.0 in one FHFMA.BF16 (exact
// product, one rounding = an fp32 add of the widened value).
__device__ __forceinline__ void acc_bf16_lo(float& a, uint32_t u) {
  asm("{.reg .b16 l, h;\n\tmov.b32 {l, h}, %1;\n\tfma.rn.f32.bf16 %0, l, %2, %0;\n\t}"
      : "+f"(a) : "r"(u), "h"((unsigned short)0x3F80));
}
__device__ __forceinline__ void acc_bf16_hi(float& a, uint32_t u) {
  asm("{.reg .b16 l, h;\n\tmov.b32 {l, h}, %1;\n\tfma.rn.f32.bf16 %0, h, %2, %0;\n\t}"
      : "+f"(a) : "r"(u), "h"((unsigned short)0x3F80));
}

// FACT: the adjacency factors as â_ij = s_i·s_j (GCN normalisation, checked at
// rdm_set_graph) and the slice was stored as bf16(s_j·X_j): the row sum needs
// no values (no val stream, no shuffles of it) and s_i is applied in the
// epilogue (Epi::rscale).
template <int G, int V, int U, bool FACT = false>
__device__ __forceinline__ void warp_nnz_range_bf(const int32_t* __restrict__ col,
                                                  const float* __restrict__ val,
                                                  const __nv_bfloat16* __restrict__ xb, int64_t ldx,
                                                  int64_t beg, int64_t end, int lane, int c8n,
                                                  float4 (&acc)[V][2]) {
  constexpr int NG = 32 / G;
  const int g = lane / G, sub = lane % G;
#pragma unroll
  for (int v = 0; v < V; ++v) acc[v][0] = acc[v][1] = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t base = beg; base < end; base += 32) {
    const int64_t j = base + lane;
    int c = 0;
    float a = 0.f;
    if (j < end) {
      c = __ldcs(col + j);
      if (!FACT) a = __ldcs(val + j);
    }
    const int cnt = (end - base) < 32 ? (int)(end - base) : 32;
#pragma unroll
    for (int t0 = 0; t0 < G; t0 += U) {
      if (t0 * NG >= cnt) break;   // warp-uniform: the rest of the batch is past the row's end
      uint4 x[U][V];
      float vv[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int k = (t0 + u) * NG + g;
        const int cc = (G == 1) ? c : __shfl_sync(kFull, c, k);
        vv[u] = FACT ? 1.f : (G == 1) ? a : __shfl_sync(kFull, a, k);
        const uint4* xr = reinterpret_cast<const uint4*>(xb + (int64_t)cc * ldx);
#pragma unroll
        for (int v = 0; v < V; ++v)
          x[u][v] = (k < cnt && v * G + sub < c8n) ? RDM_GATHER_LD(xr + v * G + sub) : make_uint4(0u, 0u, 0u, 0u);
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          const uint32_t w4[4] = {x[u][v].x, x[u][v].y, x[u][v].z, x[u][v].w};
          if constexpr (FACT) {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              acc_bf16_lo(acc[v][h].x, w4[2 * h]);
              acc_bf16_hi(acc[v][h].y, w4[2 * h]);
              acc_bf16_lo(acc[v][h].z, w4[2 * h + 1]);
              acc_bf16_hi(acc[v][h].w, w4[2 * h + 1]);
            }
          } else {
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              float4& A = acc[v][h];
              A.x = fmaf(vv[u], __uint_as_float(w4[2 * h] << 16), A.x);
              A.y = fmaf(vv[u], __uint_as_float(w4[2 * h] & 0xFFFF0000u), A.y);
              A.z = fmaf(vv[u], __uint_as_float(w4[2 * h + 1] << 16), A.z);
              A.w = fmaf(vv[u], __uint_as_float(w4[2 * h + 1] & 0xFFFF0000u), A.w);
            }
          }
        }
    }
  }
#pragma unroll
  for (int off = G; off < 32; off <<= 1) {
#pragma unroll
    for (int v = 0; v < V; ++v)
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        acc[v][h].x += __shfl_xor_sync(kFull, acc[v][h].x, off);
        acc[v][h].y += __shfl_xor_sync(kFull, acc[v][h].y, off);
        acc[v][h].z += __shfl_xor_sync(kFull, acc[v][h].z, off);
        acc[v][h].w += __shfl_xor_sync(kFull, acc[v][h].w, off);
      }
  }
}

// bf16 variant of spmm_kernel (same items, bins and epilogue); a vector is 8
// columns, `w4` is the output's real padded width (stores stop there).
// twice the accumulators of spmm_kernel: s = 2V + U·V slots
constexpr int spmm_minb_bf(int V, int U) { return spmm_minb_slots(2 * V + U * V); }
template <int G, int V, int U, bool FACT = false>
__global__ void __launch_bounds__(kWarps * 32, spmm_minb_bf(V, U))
spmm_kernel_bf(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
               const float* __restrict__ val, const int32_t* __restrict__ light_rows,
               const int64_t* __restrict__ seg_start, const int32_t* __restrict__ seg_row,
               int64_t n_light, int64_t n_seg, const __nv_bfloat16* __restrict__ X, int64_t ldx,
               float* __restrict__ out, int64_t ld_out, float* __restrict__ part, int64_t ld_part,
               int64_t w4, int64_t w8, int chunk8, Epi epi) {
  const int lane = threadIdx.x & 31;
  const int64_t item = (int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5);
  if (item >= n_seg + n_light) return;
  const int64_t cbase = (int64_t)blockIdx.y * chunk8 * 8;
  const int64_t rem8 = (w8 - cbase) / 8;
  const int c8n = rem8 < chunk8 ? (int)rem8 : chunk8;
  const int sub = lane % G;
  float4 acc[V][2];
  if (item < n_seg) {
    const int32_t r = seg_row[item];
    const int64_t beg = seg_start[item];
    const int64_t end = min(beg + kSeg, rowptr[r + 1]);
    warp_nnz_range_bf<G, V, U, FACT>(col, val, X + cbase, ldx, beg, end, lane, c8n, acc);
    if (lane < G) {
      float* dst = part + item * ld_part + cbase;
#pragma unroll
      for (int v = 0; v < V; ++v)
        if (v * G + sub < c8n) {
          reinterpret_cast<float4*>(dst)[2 * (v * G + sub)] = acc[v][0];
          reinterpret_cast<float4*>(dst)[2 * (v * G + sub) + 1] = acc[v][1];
        }
    }
  } else {
    const int32_t r = light_rows[item - n_seg];
    warp_nnz_range_bf<G, V, U, FACT>(col, val, X + cbase, ldx, rowptr[r], rowptr[r + 1], lane, c8n, acc);
    if (lane < G) {
      float* dst = out + (int64_t)r * ld_out;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const int ch = v * G + sub;
        if (ch < c8n) {
#pragma unroll
          for (int h = 0; h < 2; ++h) {
            const int64_t c = cbase + 8 * ch + 4 * h;
            if (c < w4) {
              const float4 o = apply_epi(acc[v][h], epi, r, c);
              *reinterpret_cast<float4*>(dst + c) = o;
              if (epi.scat.P) scatter_row_store(epi.scat, r, c, o);
            }
          }
        }
      }
    }
  }
}

// bf16 variant of spmm_short_kernel (RDM_PREC_FAST): a group of G lanes per
// short row, the row's first 32 (col, val) loaded up front and shuffled, U
// entries in flight, each lane V 128-bit gathers of 8 bf16 columns; the same
// epilogue and stores as spmm_kernel_bf.
template <int G, int V, int U, bool FACT>
__global__ void __launch_bounds__(kWarps * 32)
spmm_short_kernel_bf(const int64_t* __restrict__ rowptr, const int32_t* __restrict__ col,
                     const float* __restrict__ val, const int32_t* __restrict__ rows, int64_t n_rows,
                     const __nv_bfloat16* __restrict__ X, int64_t ldx, float* __restrict__ out, int64_t ld_out,
                     int64_t w4, int64_t w8, int chunk8, Epi epi) {
  constexpr int R = 32 / G, NB = 32, SL = NB / G;
  const int lane = threadIdx.x & 31;
  const int g = lane / G, sub = lane % G;
  const int64_t idx = ((int64_t)blockIdx.x * kWarps + (threadIdx.x >> 5)) * R + g;
  const int64_t cbase = (int64_t)blockIdx.y * chunk8 * 8;
  const int64_t rem8 = (w8 - cbase) / 8;
  const int c8n = rem8 < chunk8 ? (int)rem8 : chunk8;
  const bool live = idx < n_rows;
  const int32_t r = live ? rows[idx] : 0;
  const int64_t beg = live ? rowptr[r] : 0, end = live ? rowptr[r + 1] : 0;
  const __nv_bfloat16* xb = X + cbase;
  float4 acc[V][2];
#pragma unroll
  for (int v = 0; v < V; ++v) acc[v][0] = acc[v][1] = make_float4(0.f, 0.f, 0.f, 0.f);
  int pc[SL];
  float pv[SL];
#pragma unroll
  for (int s = 0; s < SL; ++s) {
    const int64_t j = beg + s * G + sub;
    const bool ok = j < end;
    pc[s] = ok ? __ldcs(col + j) : 0;
    pv[s] = (ok && !FACT) ? __ldcs(val + j) : 0.f;
  }
  const int deg = (int)(end - beg);
  const int dmax = __reduce_max_sync(kFull, deg < NB ? deg : NB);
  auto step = [&](const int (&c)[U], const float (&a)[U], const bool (&ok)[U]) {
    uint4 x[U][V];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v)
        x[u][v] = (ok[u] && v * G + sub < c8n)
                      ? RDM_GATHER_LD(reinterpret_cast<const uint4*>(xb + (int64_t)c[u] * ldx) + v * G + sub)
                      : make_uint4(0u, 0u, 0u, 0u);
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const uint32_t w4r[4] = {x[u][v].x, x[u][v].y, x[u][v].z, x[u][v].w};
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          float4& A = acc[v][h];
          if constexpr (FACT) {
            acc_bf16_lo(A.x, w4r[2 * h]);
            acc_bf16_hi(A.y, w4r[2 * h]);
            acc_bf16_lo(A.z, w4r[2 * h + 1]);
            acc_bf16_hi(A.w, w4r[2 * h + 1]);
          } else {
            A.x = fmaf(a[u], __uint_as_float(w4r[2 * h] << 16), A.x);
            A.y = fmaf(a[u], __uint_as_float(w4r[2 * h] & 0xFFFF0000u), A.y);
            A.z = fmaf(a[u], __uint_as_float(w4r[2 * h + 1] << 16), A.z);
            A.w = fmaf(a[u], __uint_as_float(w4r[2 * h + 1] & 0xFFFF0000u), A.w);
          }
        }
      }
  };
#pragma unroll
  for (int e0 = 0; e0 < NB; e0 += U) {
    if (e0 >= dmax) break;   // warp-uniform
    int c[U];
    float a[U];
    bool ok[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int e = e0 + u;
      c[u] = __shfl_sync(kFull, pc[e / G], g * G + (e % G));
      a[u] = FACT ? 1.f : __shfl_sync(kFull, pv[e / G], g * G + (e % G));
      ok[u] = e < deg;
    }
    step(c, a, ok);
  }
  for (int64_t j = beg + NB; j < end; j += U) {   // rows above the batch (RDM_SPMM_SHORT > 32)
    int c[U];
    float a[U];
    bool ok[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      ok[u] = j + u < end;
      c[u] = ok[u] ? __ldcs(col + j + u) : 0;
      a[u] = (ok[u] && !FACT) ? __ldcs(val + j + u) : 0.f;
    }
    step(c, a, ok);
  }
  if (!live) return;
  float* dst = out + (int64_t)r * ld_out;
#pragma unroll
  for (int v = 0; v < V; ++v) {
    const int ch = v * G + sub;
    if (ch < c8n) {
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int64_t cc = cbase + 8 * ch + 4 * h;
        if (cc < w4) {
          const float4 o = apply_epi(acc[v][h], epi, r, cc);
          *reinterpret_cast<float4*>(dst + cc) = o;
          if (epi.scat.P) scatter_row_store(epi.scat, r, cc, o);
        }
      }
    }
  }
}

// fp32 slice → bf16 copy (round to nearest even) of X (scale == null) or of
// s_r·X_r (factored adjacency), row length ldy = w8, zero pads: one thread
// per 8 columns.
__global__ void to_bf16_kernel(const float* __restrict__ X, int64_t ldx, int64_t n, int64_t w4, int64_t w8,
                               __nv_bfloat16* __restrict__ Y, const float* __restrict__ scale) {
  const int64_t per = w8 / 8;
  const int64_t total = n * per;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / per, c = (i - r * per) * 8;
    const float* xr = X + r * ldx + c;
    float4 a = __ldcs(reinterpret_cast<const float4*>(xr));
    float4 b = (c + 4 < w4) ? __ldcs(reinterpret_cast<const float4*>(xr + 4)) : make_float4(0.f, 0.f, 0.f, 0.f);
    if (scale) {
      const float sc = __ldg(scale + r);
      a.x *= sc; a.y *= sc; a.z *= sc; a.w *= sc;
      b.x *= sc; b.y *= sc; b.z *= sc; b.w *= sc;
    }
    __nv_bfloat162 p[4] = {__floats2bfloat162_rn(a.x, a.y), __floats2bfloat162_rn(a.z, a.w),
                           __floats2bfloat162_rn(b.x, b.y), __floats2bfloat162_rn(b.z, b.w)};
    *reinterpret_cast<uint4*>(Y + r * w8 + c) = *reinterpret_cast<const uint4*>(p);
  }
}

// Heavy rows: sum the partial rows of their segments in segment order.
__global__ void spmm_heavy_reduce(const int32_t* __restrict__ heavy_rows,
                                  const int32_t* __restrict__ heavy_seg,
                                  const float* __restrict__ part, int64_t ld_part,
                                  float* __restrict__ out, int64_t ld_out, int64_t w4, Epi epi) {
  const int64_t h = blockIdx.x;
  const int32_t r = heavy_rows[h];
  const int s0 = heavy_seg[h], s1 = heavy_seg[h + 1];
  for (int64_t c = (int64_t)threadIdx.x * 4; c < w4; c += (int64_t)blockDim.x * 4) {
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    for (int s = s0; s < s1; ++s) {
      const float4 p = *reinterpret_cast<const float4*>(part + (int64_t)s * ld_part + c);
      acc.x += p.x; acc.y += p.y; acc.z += p.z; acc.w += p.w;
    }
    const float4 o = apply_epi(acc, epi, r, c);
    *reinterpret_cast<float4*>(out + (int64_t)r * ld_out + c) = o;
    if (epi.scat.P) scatter_row_store(epi.scat, r, c, o);
  }
}

template <int G, int V, int U>
void launch_spmm(rdm_ctx* ctx, const Csr& A, const float* in, int64_t ld_in, float* out,
                 int64_t ld_out, float* part, int64_t ld_part, int64_t w4, int chunk4,
                 const Epi& epi, const Hot& hot, int64_t n_long) {
  const int64_t items = A.n_seg + n_long;
  if (items == 0) return;
  const int64_t chunks = ceil_div(w4, 4 * chunk4);
  dim3 grid((unsigned)ceil_div(items, kWarps), (unsigned)chunks);
  spmm_kernel<G, V, U><<<grid, kWarps * 32, 0, ctx->stream>>>(
      A.rowptr->as<int64_t>(), hot.hw ? A.col_hot->as<int32_t>() : A.col->as<int32_t>(), A.val->as<float>(),
      A.light_rows->as<int32_t>(), A.seg_start->as<int64_t>(),
      reinterpret_cast<const int32_t*>(A.seg_start->as<int64_t>() + A.n_seg), n_long, A.n_seg,
      hot.hw ? hot.xh : in, hot.hw ? hot.ldh : ld_in, out, ld_out, part, ld_part, w4, chunk4, epi);
  RDM_LAUNCHED(ctx);
}

// The short light rows [n_long, n_light) of the light-row list.
template <int G, int V, int U>
void launch_spmm_short(rdm_ctx* ctx, const Csr& A, const float* in, int64_t ld_in, float* out, int64_t ld_out,
                       int64_t w4, int chunk4, const Epi& epi, const Hot& hot, int64_t n_long,
                       cudaStream_t st, int short_deg) {
  const int64_t n_short = A.n_light - n_long;
  if (n_short <= 0) return;
  constexpr int R = 32 / G;
  const int64_t chunks = ceil_div(w4, 4 * chunk4);
  dim3 grid((unsigned)ceil_div(n_short, (int64_t)kWarps * R), (unsigned)chunks);
  auto kern = short_deg > 32 ? spmm_short_kernel<G, V, U, 64> : spmm_short_kernel<G, V, U, 32>;
  kern<<<grid, kWarps * 32, 0, st>>>(
      A.rowptr->as<int64_t>(), hot.hw ? A.col_hot->as<int32_t>() : A.col->as<int32_t>(), A.val->as<float>(),
      A.light_rows->as<int32_t>() + n_long, n_short, hot.hw ? hot.xh : in, hot.hw ? hot.ldh : ld_in, out, ld_out,
      w4, chunk4, epi);
  RDM_LAUNCHED(ctx);
}

template <int G, int V, int U, bool FACT = false>
void launch_spmm_bf(rdm_ctx* ctx, const Csr& A, const __nv_bfloat16* in, int64_t ld_in, float* out,
                    int64_t ld_out, float* part, int64_t ld_part, int64_t w4, int64_t w8, int chunk8,
                    const Epi& epi, int64_t n_long = -1) {
  if (n_long < 0) n_long = A.n_light;
  const int64_t items = A.n_seg + n_long;
  if (items == 0) return;
  const int64_t chunks = ceil_div(w8, 8 * chunk8);
  dim3 grid((unsigned)ceil_div(items, kWarps), (unsigned)chunks);
  spmm_kernel_bf<G, V, U, FACT><<<grid, kWarps * 32, 0, ctx->stream>>>(
      A.rowptr->as<int64_t>(), A.col->as<int32_t>(), A.val->as<float>(),
      A.light_rows->as<int32_t>(), A.seg_start->as<int64_t>(),
      reinterpret_cast<const int32_t*>(A.seg_start->as<int64_t>() + A.n_seg), n_long, A.n_seg,
      in, ld_in, out, ld_out, part, ld_part, w4, w8, chunk8, epi);
  RDM_LAUNCHED(ctx);
}

// The short light rows [n_long, n_light) of the bf16 path (2 entries in flight).
template <int G, int V, bool FACT>
void launch_spmm_short_bf(rdm_ctx* ctx, const Csr& A, const __nv_bfloat16* in, int64_t ld_in, float* out,
                          int64_t ld_out, int64_t w4, int64_t w8, int chunk8, const Epi& epi, int64_t n_long,
                          cudaStream_t st) {
  const int64_t n_short = A.n_light - n_long;
  if (n_short <= 0) return;
  constexpr int R = 32 / G;
  const int64_t chunks = ceil_div(w8, 8 * chunk8);
  dim3 grid((unsigned)ceil_div(n_short, (int64_t)kWarps * R), (unsigned)chunks);
  spmm_short_kernel_bf<G, V, 2, FACT><<<grid, kWarps * 32, 0, st>>>(
      A.rowptr->as<int64_t>(), A.col->as<int32_t>(), A.val->as<float>(), A.light_rows->as<int32_t>() + n_long,
      n_short, in, ld_in, out, ld_out, w4, w8, chunk8, epi);
  RDM_LAUNCHED(ctx);
}

// (G, V) for a chunk of c4 float4 columns: fewest lane slots G·V ≥ c4, ties to
// the G closest to 8 (short reductions, several nnz in flight).
void pick_gv(int c4, int* G, int* V) {
  int best_s = 1 << 30, bg = 32, bv = 1;
  for (int v = 1; v <= 4; ++v) {
    int g = 1;
    while (g * v < c4) g <<= 1;
    if (g > 32) continue;
    const int s = g * v;
    const int d = g > 8 ? g / 8 : 8 / g, bd = bg > 8 ? bg / 8 : 8 / bg;
    if (s < best_s || (s == best_s && d < bd)) {
      best_s = s;
      bg = g;
      bv = v;
    }
  }
  *G = bg;
  *V = bv;
}

void run_csr(rdm_ctx* ctx, const Csr& A, const float* in, int64_t ld_in, float* out, int64_t ld_out,
             int64_t w4, const Epi& epi, const __nv_bfloat16* inb, bool fact = false);

// (G, V, U) for a chunk of c 128-bit vectors per row (4 fp32 or 8 bf16
// columns each).  Measured on the Reddit- and products-shaped residual CSRs
// (tools/exp_gvu.py, profiles/r1_spmm_gvu.txt): for bf16 rows several nnz in
// flight per group (U) pay; fp32 keeps U = 1 (best or tied at every width).
void pick_gvu(int c, bool bf, int* G, int* V, int* U, bool dram_slice = false, bool near_l2 = false) {
  pick_gv(c, G, V);
  *U = 1;
  if (!bf) {
    // 9-12 vectors (w = 33..48): 8 lanes x 2 (profiles/r2_spmm_gvu.txt: w = 41 0.82 → 0.79 ms)
    if (c >= 9 && c <= 12) { *G = 8; *V = 2; }
    // slices of 17-32 vectors up to ≈ 2 L2s (Reddit-shaped w = 128, 119 MB):
    // 16 lanes x 2 — fewer registers, 6 CTAs per SM instead of 4 (1.207 →
    // 1.168 ms per call, profiles/r2_spmm_u.txt)
    if (near_l2 && c >= 17 && c <= 32) { *G = 16; *V = 2; }
    // DRAM-resident slices of 5-8 vectors (products-shaped w = 32 at P = 8):
    // 4 nnz in flight per group (2.61 → 2.46 ms); at <= 4 vectors U = 1 stays
    // best (papers100M-shaped w = 16: U = 4 85 ms vs U = 1 77 ms, r2_relabel.md)
    if (dram_slice && c >= 5 && c <= 8) { *V = 1; *G = 8; *U = 4; }
  }
  if (bf) {
    if (c >= 3 && c <= 8) { *G = 8; *V = 1; *U = 4; }
    else if (c >= 9 && c <= 16) { *G = 8; *V = 2; *U = 2; }
    else if (c >= 17 && c <= 32) { *G = 16; *V = 2; *U = 2; }
    else if (c <= 2) *U = std::min(*G, 2);
  }   // fp32: U = 1 measured best or tied at every width
}

// Hub-core cost model (B200-calibrated, profiles/r1_core_experiment.md): the
// CSR SpMM spends ≈ 24 ps · (w/128)^0.55 per nnz (L2-gather bound), the core
// GEMM ≈ 1.25 ps per K² element (A-operand stream + 3xTF32 MMA), both per call.
double core_saving_s(int64_t core_nnz, int64_t w) {
  return (double)core_nnz * 24e-12 * std::pow((double)w / 128.0, 0.55);
}
double core_cost_s(int64_t K, int64_t w) { return (double)K * K * 1.25e-12 * (1.0 + w / 600.0) + 20e-6; }
bool core_pays(const Core& c, int64_t w) {
  return c.forced || core_saving_s(c.nnz, w) > core_cost_s(c.K, w);
}

}  // namespace

// Core size (multiple of 128, <= kmax) with the largest modelled saving at the
// reference width 128, at least 0.1 ms per call; bucket[b] = entries whose
// larger endpoint degree-rank lies in [128 b, 128 b + 128).  `force` (an env
// value, tests): use that size.  0 = no core.
int64_t choose_core_K(const int64_t* bucket, int64_t kmax, const char* force, bool* forced) {
  int64_t best_K = 0;
  double best_gain = 1e-4;
  int64_t acc = 0;
  for (int64_t K = 128; K <= kmax; K += 128) {
    acc += bucket[K / 128 - 1];
    const double gain = core_saving_s(acc, 128) - core_cost_s(K, 128);
    if (gain > best_gain) {
      best_gain = gain;
      best_K = K;
    }
  }
  *forced = false;
  if (force && atoi(force) > 0 && kmax >= 128) {
    best_K = std::min<int64_t>(kmax, std::max<int64_t>(128, (int64_t)atoi(force) / 128 * 128));
    *forced = true;
  }
  return best_K;
}

namespace {
// Panels of X[hubs] for the core GEMM: Bt_hi/lo[n][k] = tf32 split of X[hub_ids[k]][n]
// (transposed through shared memory: coalesced reads along n, writes along k).
__global__ void core_panels_kernel(const float* __restrict__ X, int64_t ldx,
                                   const int32_t* __restrict__ hub_ids, int64_t K, int64_t w,
                                   float* __restrict__ bhi, float* __restrict__ blo) {
  __shared__ float t[32][33];
  const int64_t k0 = (int64_t)blockIdx.x * 32, n0 = (int64_t)blockIdx.y * 32;
  for (int i = threadIdx.y; i < 32; i += 8) {
    const int64_t k = k0 + i, n = n0 + threadIdx.x;
    t[i][threadIdx.x] = (n < w) ? X[(int64_t)hub_ids[k] * ldx + n] : 0.f;
  }
  __syncthreads();
  for (int i = threadIdx.y; i < 32; i += 8) {
    const int64_t n = n0 + i, k = k0 + threadIdx.x;
    if (n < w) {
      const float x = t[threadIdx.x][i];
      const float h = tf32_rn(x);
      bhi[n * K + k] = h;
      blo[n * K + k] = tf32_rn(x - h);
    }
  }
}

}  // namespace

void spmm(rdm_ctx* ctx, const Csr& A, const float* in, int64_t ld_in, float* out, int64_t ld_out,
          int64_t w, int epi_flags, const float* bias, const float* mask, int64_t ld_mask,
          const Scatter* scat) {
  RDM_CHECK_ARG(w >= 0, "spmm: negative width");
  if (w == 0 || A.n == 0) return;
  const int64_t w4 = roundup4(w);
  RDM_CHECK_ARG(ld_in >= w4 && ld_out >= w4 && ld_in % 4 == 0 && ld_out % 4 == 0,
                "spmm: leading dims must be multiples of 4 and >= roundup4(w)");
  RDM_CHECK_ARG(((uintptr_t)in & 15) == 0 && ((uintptr_t)out & 15) == 0,
                "spmm: in/out must be 16-byte aligned");
  RDM_CHECK_ARG(!(epi_flags & RDM_EPI_MASK) || (mask && ld_mask >= w4 && ld_mask % 4 == 0 &&
                                                ((uintptr_t)mask & 15) == 0),
                "spmm: mask requires a 16-byte aligned N x w buffer with ld % 4 == 0");
  RDM_CHECK_ARG(!(epi_flags & RDM_EPI_BIAS) || bias, "spmm: bias pointer missing");
  Epi epi{epi_flags, bias, mask, ld_mask, w, nullptr, 0, nullptr, nullptr, 0, nullptr, 7, nullptr, Scatter{}, nullptr};
  if (scat) {
    RDM_CHECK_ARG(scat->mode == 2 && scat->P >= 1 && scat->P <= Scatter::kMax && scat->my_w <= w,
                  "spmm: bad scatter descriptor");
    epi.scat = *scat;
  }
  // RDM_PREC_FAST: one bf16 copy of the input slice per call, gathered by
  // every row of the residual CSR (rdm.h rdm_set_precision)
  const __nv_bfloat16* inb = nullptr;
  bool fact = false;
  if (ctx->prec == RDM_PREC_FAST) {
    const int64_t w8 = (w4 + 7) & ~int64_t(7);
    const int64_t nin = A.in_rows();
    __nv_bfloat16* xb = reinterpret_cast<__nv_bfloat16*>(ensure_ws(ctx->ws_bf16, (size_t)std::max<int64_t>(nin, 1) * w8 * 2));
    if (ctx->bf16_twin_src == in) {
      // the producing GEMM already wrote this bf16 input (cast folded into its epilogue)
      fact = ctx->bf16_twin_fact;
    } else {
      const int64_t total = nin * (w8 / 8);
      const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(total, 256), (int64_t)ctx->num_sms * 16));
      // the value-free factored rows need bf16(s_j·X_j); an input that already
      // holds bf16 values (bf16 wire) is used as is, with the values (no second rounding)
      fact = A.fscale != nullptr && !ctx->spmm_in_bf16;
      to_bf16_kernel<<<grid, 256, 0, ctx->stream>>>(in, ld_in, nin, w4, w8, xb,
                                                    fact ? A.fscale->as<float>() : nullptr);
      RDM_LAUNCHED(ctx);
    }
    ctx->bf16_twin_src = nullptr;
    inb = xb;
    if (fact) epi.rscale = A.fscale->as<float>();
  }
  // hub-tile pieces: 2 column-scaled fp16 pieces (fp32-class, default), 3 bf16
  // pieces (RDM_TILE_PIECES=3, the earlier form) or 1 bf16 piece (fast)
  // (measured, tools/exp_tiles.py: fp16 pairs pay where the tile is MMA-bound,
  // w > 64: 1.53 → 1.44 ms at w = 128; narrower tiles are bound by the bit
  // expansion and the extra column-max pass makes fp16 pairs slower)
  int np = ctx->prec == RDM_PREC_FAST ? kPiecesI8x2 : kPiecesI8;
  if (ctx->prec == RDM_PREC_FAST)
    if (const char* e = getenv("RDM_TILE_PIECES_FAST")) np = atoi(e) == 1 ? 1 : kPiecesI8x2;
  if (ctx->prec != RDM_PREC_FAST)
    if (const char* e = getenv("RDM_TILE_PIECES")) np = atoi(e) == 3 ? 3 : atoi(e) == 2 ? 2 : kPiecesI8;
  if (A.core.n_tiles && hub_tiles_pay(A.core, w, np)) {
    // binary hub tiles on the kind::f16 tensor cores (hubtiles.cu); the
    // residual CSR's epilogue adds s_i · Σ_items partial for hub rows.
    const int64_t ldp = w4;
    const bool pairs = (np == kPiecesI8 || np == kPiecesI8x2) && tiles_paired();
    const size_t prow = pairs ? (size_t)A.core.n_pitems * 256 : (size_t)A.core.n_items * 128;
    float* part = ensure_ws(ctx->ws_core_c, prow * ldp * sizeof(float));
    hub_tiles_product(ctx, A.core, in, ld_in, w, part, ldp, np);
    epi.tpart = part;
    epi.ld_tpart = ldp;
    epi.rb_item = pairs ? A.core.pair_item->as<int32_t>() : A.core.rb_item->as<int32_t>();
    epi.item_shift = pairs ? 8 : 7;
    epi.tscale = A.core.rscale->as<float>();
    epi.hub_slot = A.core.hub_slot->as<int32_t>();
    run_csr(ctx, *A.core.resid, in, ld_in, out, ld_out, w4, epi, inb, fact);
  } else if (A.core.K && core_pays(A.core, w)) {
    // hub core on the tensor cores: panels Bt[n][k] = split(X[hub_k][n]), then
    // C_core = Acore · X[hubs]; the residual CSR's epilogue adds C_core rows.
    const int64_t K = A.core.K;
    float* bp = ensure_ws(ctx->ws_core_b, (size_t)2 * w * K * sizeof(float));
    float* cc = ensure_ws(ctx->ws_core_c, (size_t)K * w4 * sizeof(float));
    dim3 grid((unsigned)(K / 32), (unsigned)ceil_div(w, 32));
    core_panels_kernel<<<grid, dim3(32, 8), 0, ctx->stream>>>(in, ld_in, A.core.hub_ids->as<int32_t>(),
                                                              K, w, bp, bp + w * K);
    RDM_LAUNCHED(ctx);
    gemm_tc_panels(ctx, A.core.A->as<float>(), K, bp, bp + w * K, K, cc, w4, K, w, K);
    epi.core = cc;
    epi.ld_core = w4;
    epi.hub_slot = A.core.hub_slot->as<int32_t>();
    run_csr(ctx, *A.core.resid, in, ld_in, out, ld_out, w4, epi, inb, fact);
  } else {
    run_csr(ctx, A, in, ld_in, out, ld_out, w4, epi, inb, fact);
  }
  ctx->counters.spmm_calls++;
  ctx->counters.spmm_nnz_cols += A.nnz * w;
}

namespace {
// X'[r] = X[ids[r]] (float4 copies, full leading dim).
__global__ void rank_gather_kernel(const float* __restrict__ X, int64_t ldx, const int32_t* __restrict__ ids,
                                   int64_t n, int64_t ld4, float* __restrict__ xh) {
  const int64_t total = n * ld4;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / ld4, c = i - r * ld4;
    reinterpret_cast<float4*>(xh)[i] = __ldg(reinterpret_cast<const float4*>(X + (int64_t)__ldg(ids + r) * ldx) + c);
  }
}

// Per call: the input slice in rank order (one gather pass, 2·N·ld·4 bytes).
Hot rank_panel(rdm_ctx* ctx, const Csr& A, const float* in, int64_t ld_in) {
  const int64_t n = A.hot_max;
  float* xh = ensure_ws(ctx->ws_hot, (size_t)n * ld_in * sizeof(float));
  const int64_t total = n * (ld_in / 4);
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(total, 256), (int64_t)ctx->num_sms * 16));
  rank_gather_kernel<<<grid, 256, 0, ctx->stream>>>(in, ld_in, A.hot_ids->as<int32_t>(), n, ld_in / 4, xh);
  RDM_LAUNCHED(ctx);
  return Hot{xh, ld_in, 1};
}

void run_csr(rdm_ctx* ctx, const Csr& A, const float* in, int64_t ld_in, float* out, int64_t ld_out,
             int64_t w4, const Epi& epi, const __nv_bfloat16* inb, bool fact) {
  const int64_t w8 = (w4 + 7) & ~int64_t(7);
  const int64_t ldp = inb ? w8 : w4;
  float* part = nullptr;
  if (A.n_seg) part = ensure_ws(ctx->ws_seg, (size_t)A.n_seg * ldp * sizeof(float));
  int G, V;
  // Column chunks (blockIdx.y, scheduled chunk after chunk): narrower chunks
  // keep the gathered slice L2-resident at the price of re-streaming the CSR.
  // Measured (profiles/r1_summary.md): one 256-wide chunk beats two 128-wide
  // ones for 128 < w <= 256 (the CSR is streamed once); wider slices use
  // 128-wide chunks; narrower chunks lose more to CSR re-streaming than they
  // gain in L2 residency.
  int chunk4 = (w4 > 128 && w4 <= 256) ? 64 : 32;
  if (const char* e = getenv("RDM_SPMM_CHUNK4")) chunk4 = std::max(1, std::min(64, atoi(e)));
  // U = nnz gathered per group before use (loads in flight); the default
  // keeps ≈ 4 loads of 16 B in flight per lane
  if (const char* e = getenv("RDM_SPMM_GV")) {   // experiments: "G,V"
    G = atoi(e);
    const char* c = strchr(e, ',');
    V = c ? atoi(c + 1) : 1;
  }
  if (inb) {
    // bf16 rows: the same column chunks, 8 columns per 128-bit gather
    const int chunk8 = std::max(1, chunk4 / 2);
    const int c8 = (int)std::min<int64_t>(chunk8, w8 / 8);
    int U = 1;
    if (!getenv("RDM_SPMM_GV")) pick_gvu(c8, true, &G, &V, &U);
    if (const char* e = getenv("RDM_SPMM_U")) U = atoi(e);
    // short light rows (degree ≤ 32) on the auxiliary stream, as in the fp32 path
    // (RDM_SPMM_SHORT_BF=0: warp-per-row for every light row)
    const char* sbf = getenv("RDM_SPMM_SHORT_BF");
    int64_t n_long = A.n_light;
    bool fork = false;
    if (!(sbf && !atoi(sbf))) {
      int sg, sv;
      pick_gv(c8, &sg, &sv);
      const int64_t nl = A.deg_ge[33 <= Csr::kDegTab ? 33 : Csr::kDegTab];
      if (A.n_light > nl) {
        if (!ctx->aux) {
          int lo = 0, hi = 0;
          RDM_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
          RDM_CUDA(cudaStreamCreateWithPriority(&ctx->aux, cudaStreamNonBlocking, lo));
          RDM_CUDA(cudaEventCreateWithFlags(&ctx->aux_fork, cudaEventDisableTiming));
          RDM_CUDA(cudaEventCreateWithFlags(&ctx->aux_join, cudaEventDisableTiming));
        }
        RDM_CUDA(cudaEventRecord(ctx->aux_fork, ctx->stream));
        RDM_CUDA(cudaStreamWaitEvent(ctx->aux, ctx->aux_fork, 0));
        bool done = true;
#define RDM_SHORT_BF_CASE(g_, v_)                                                                       \
  if (sg == g_ && sv == v_) {                                                                           \
    if (fact) launch_spmm_short_bf<g_, v_, true>(ctx, A, inb, w8, out, ld_out, w4, w8, chunk8, epi, nl, ctx->aux); \
    else launch_spmm_short_bf<g_, v_, false>(ctx, A, inb, w8, out, ld_out, w4, w8, chunk8, epi, nl, ctx->aux);     \
  } else
        RDM_SHORT_BF_CASE(1, 1) RDM_SHORT_BF_CASE(2, 1) RDM_SHORT_BF_CASE(2, 2) RDM_SHORT_BF_CASE(2, 3)
        RDM_SHORT_BF_CASE(4, 1) RDM_SHORT_BF_CASE(4, 2) RDM_SHORT_BF_CASE(4, 3) RDM_SHORT_BF_CASE(4, 4)
        RDM_SHORT_BF_CASE(8, 1) RDM_SHORT_BF_CASE(8, 2) RDM_SHORT_BF_CASE(8, 3) RDM_SHORT_BF_CASE(8, 4)
        RDM_SHORT_BF_CASE(16, 1) RDM_SHORT_BF_CASE(16, 2) RDM_SHORT_BF_CASE(16, 3) RDM_SHORT_BF_CASE(16, 4)
        RDM_SHORT_BF_CASE(32, 1) { done = false; }
#undef RDM_SHORT_BF_CASE
        if (done) {
          n_long = nl;
          fork = true;
        }
        RDM_CUDA(cudaEventRecord(ctx->aux_join, ctx->aux));
        if (!done) RDM_CUDA(cudaStreamWaitEvent(ctx->stream, ctx->aux_join, 0));
      }
    }
    auto join = [&]() {
      if (fork) RDM_CUDA(cudaStreamWaitEvent(ctx->stream, ctx->aux_join, 0));
    };
    if (fact) {   // value-free sums of bf16(s_j X_j) for the measured mappings
#define RDM_SPMM_FCASE(g_, v_, u_) \
  if (G == g_ && V == v_ && U == u_) { launch_spmm_bf<g_, v_, u_, true>(ctx, A, inb, w8, out, ld_out, part, ldp, w4, w8, chunk8, epi, n_long); join(); fact = false; goto heavy; }
      RDM_SPMM_FCASE(8, 1, 4) RDM_SPMM_FCASE(8, 2, 2) RDM_SPMM_FCASE(16, 2, 2) RDM_SPMM_FCASE(2, 1, 2)
      RDM_SPMM_FCASE(1, 2, 1) RDM_SPMM_FCASE(1, 1, 1) RDM_SPMM_FCASE(4, 1, 2) RDM_SPMM_FCASE(32, 1, 2)
#undef RDM_SPMM_FCASE
      throw Error(RDM_ERR_STATE, "spmm: no factored bf16 kernel for G/V/U");
    }
#define RDM_SPMM_CASE(g_, v_, u_) \
  if (G == g_ && V == v_ && U == u_) launch_spmm_bf<g_, v_, u_>(ctx, A, inb, w8, out, ld_out, part, ldp, w4, w8, chunk8, epi, n_long); else
    RDM_SPMM_CASE(1, 1, 1) RDM_SPMM_CASE(1, 2, 1) RDM_SPMM_CASE(1, 3, 1) RDM_SPMM_CASE(1, 4, 1)
    RDM_SPMM_CASE(2, 1, 1) RDM_SPMM_CASE(2, 1, 2) RDM_SPMM_CASE(2, 2, 1) RDM_SPMM_CASE(2, 2, 2)
    RDM_SPMM_CASE(2, 3, 1) RDM_SPMM_CASE(2, 3, 2) RDM_SPMM_CASE(2, 4, 1) RDM_SPMM_CASE(2, 4, 2)
    RDM_SPMM_CASE(4, 1, 1) RDM_SPMM_CASE(4, 1, 2) RDM_SPMM_CASE(4, 1, 4) RDM_SPMM_CASE(4, 2, 1)
    RDM_SPMM_CASE(4, 2, 2) RDM_SPMM_CASE(4, 2, 4) RDM_SPMM_CASE(4, 3, 1) RDM_SPMM_CASE(4, 3, 2)
    RDM_SPMM_CASE(4, 4, 1) RDM_SPMM_CASE(4, 4, 2) RDM_SPMM_CASE(8, 1, 1) RDM_SPMM_CASE(8, 1, 2)
    RDM_SPMM_CASE(8, 1, 4) RDM_SPMM_CASE(8, 2, 1) RDM_SPMM_CASE(8, 2, 2) RDM_SPMM_CASE(8, 2, 4)
    RDM_SPMM_CASE(8, 3, 1) RDM_SPMM_CASE(8, 3, 2) RDM_SPMM_CASE(8, 4, 1) RDM_SPMM_CASE(8, 4, 2)
    RDM_SPMM_CASE(16, 1, 1) RDM_SPMM_CASE(16, 1, 2) RDM_SPMM_CASE(16, 1, 4) RDM_SPMM_CASE(16, 2, 1)
    RDM_SPMM_CASE(16, 2, 2) RDM_SPMM_CASE(16, 2, 4) RDM_SPMM_CASE(16, 3, 1) RDM_SPMM_CASE(16, 3, 2)
    RDM_SPMM_CASE(16, 4, 1) RDM_SPMM_CASE(16, 4, 2) RDM_SPMM_CASE(32, 1, 1) RDM_SPMM_CASE(32, 1, 2)
    RDM_SPMM_CASE(32, 1, 4)
    throw Error(RDM_ERR_ARG, "spmm: no bf16 kernel for G/V/U");
#undef RDM_SPMM_CASE
    join();
  } else {
    const int c4 = (int)std::min<int64_t>(chunk4, w4 / 4);
    int U = 1;
    const double slice_bytes = (double)A.in_rows() * (double)ld_in * 4.0;
    const bool dram_slice = slice_bytes > 96e6;
    if (!getenv("RDM_SPMM_GV")) pick_gvu(c4, false, &G, &V, &U, dram_slice, slice_bytes <= 256e6);
    Hot hot{nullptr, 0, 0};
    const char* rl = getenv("RDM_RELABEL");   // column relabelling of DRAM-resident slices (experiment)
    if (dram_slice && A.col_hot && !(rl && !atoi(rl))) hot = rank_panel(ctx, A, in, ld_in);
    // short light rows (degree <= RDM_SPMM_SHORT, default 32) → row-per-group kernel
    // degree threshold of the short-row kernel: 64 for slices up to 25 vectors
    // (w ≤ 100: w = 41 0.625 → 0.608, w = 47 2.50 → 2.41, w = 100 4.82 → 4.73
    // ms per call), 32 for wider ones (w = 256: 8.15 vs 8.72 at 64),
    // profiles/r2_spmm_short_thr.txt
    int short_deg = c4 <= 25 ? 64 : 32;
    if (const char* e = getenv("RDM_SPMM_SHORT")) short_deg = std::max(0, std::min(Csr::kDegTab, atoi(e)));
    const int64_t n_long = short_deg > 0 ? A.deg_ge[short_deg + 1 <= Csr::kDegTab ? short_deg + 1 : Csr::kDegTab]
                                         : A.n_light;
    // The short rows run on the auxiliary stream beside the long-row kernel
    // (disjoint output rows, both read only the tile partials finished
    // before): its CTAs fill the long kernel's register-limited occupancy and
    // its tail.  RDM_SPMM_CONC=0: one stream (experiments).
    const char* conc_e = getenv("RDM_SPMM_CONC");
    const bool conc = short_deg > 0 && A.n_light > n_long && (A.n_seg + n_long) > 0 && !(conc_e && !atoi(conc_e));
    cudaStream_t sst = ctx->stream;
    if (conc) {
      if (!ctx->aux) {
        int lo = 0, hi = 0;
        RDM_CUDA(cudaDeviceGetStreamPriorityRange(&lo, &hi));
        RDM_CUDA(cudaStreamCreateWithPriority(&ctx->aux, cudaStreamNonBlocking, lo));
        RDM_CUDA(cudaEventCreateWithFlags(&ctx->aux_fork, cudaEventDisableTiming));
        RDM_CUDA(cudaEventCreateWithFlags(&ctx->aux_join, cudaEventDisableTiming));
      }
      RDM_CUDA(cudaEventRecord(ctx->aux_fork, ctx->stream));
      RDM_CUDA(cudaStreamWaitEvent(ctx->aux, ctx->aux_fork, 0));
      sst = ctx->aux;
    }
    if (short_deg > 0) {
      int sg, sv;
      pick_gv(c4, &sg, &sv);
#define RDM_SHORT_CASE(g_, v_) \
  if (sg == g_ && sv == v_) launch_spmm_short<g_, v_, 2>(ctx, A, in, ld_in, out, ld_out, w4, chunk4, epi, hot, n_long, sst, short_deg); else
      RDM_SHORT_CASE(1, 1) RDM_SHORT_CASE(1, 2) RDM_SHORT_CASE(1, 3) RDM_SHORT_CASE(1, 4)
      RDM_SHORT_CASE(2, 1) RDM_SHORT_CASE(2, 2) RDM_SHORT_CASE(2, 3) RDM_SHORT_CASE(2, 4)
      RDM_SHORT_CASE(4, 1) RDM_SHORT_CASE(4, 2) RDM_SHORT_CASE(4, 3) RDM_SHORT_CASE(4, 4)
      RDM_SHORT_CASE(8, 1) RDM_SHORT_CASE(8, 2) RDM_SHORT_CASE(8, 3) RDM_SHORT_CASE(8, 4)
      RDM_SHORT_CASE(16, 1) RDM_SHORT_CASE(16, 2) RDM_SHORT_CASE(16, 3) RDM_SHORT_CASE(16, 4)
      RDM_SHORT_CASE(32, 1) RDM_SHORT_CASE(32, 2)
      throw Error(RDM_ERR_ARG, "spmm: no short-row kernel for G/V");
#undef RDM_SHORT_CASE
    }
    if (const char* e = getenv("RDM_SPMM_U")) U = atoi(e);
#define RDM_SPMM_CASE(g_, v_, u_) \
  if (G == g_ && V == v_ && U == u_) launch_spmm<g_, v_, u_>(ctx, A, in, ld_in, out, ld_out, part, w4, w4, chunk4, epi, hot, n_long); else
    RDM_SPMM_CASE(1, 1, 1) RDM_SPMM_CASE(1, 2, 1) RDM_SPMM_CASE(1, 3, 1) RDM_SPMM_CASE(1, 4, 1)
    RDM_SPMM_CASE(2, 1, 1) RDM_SPMM_CASE(2, 1, 2) RDM_SPMM_CASE(2, 2, 1) RDM_SPMM_CASE(2, 2, 2)
    RDM_SPMM_CASE(2, 3, 1) RDM_SPMM_CASE(2, 3, 2) RDM_SPMM_CASE(2, 4, 1) RDM_SPMM_CASE(2, 4, 2)
    RDM_SPMM_CASE(4, 1, 1) RDM_SPMM_CASE(4, 1, 2) RDM_SPMM_CASE(4, 1, 4) RDM_SPMM_CASE(4, 2, 1)
    RDM_SPMM_CASE(4, 2, 2) RDM_SPMM_CASE(4, 2, 4) RDM_SPMM_CASE(4, 3, 1) RDM_SPMM_CASE(4, 3, 2)
    RDM_SPMM_CASE(4, 4, 1) RDM_SPMM_CASE(4, 4, 2) RDM_SPMM_CASE(8, 1, 1) RDM_SPMM_CASE(8, 1, 2)
    RDM_SPMM_CASE(8, 1, 4) RDM_SPMM_CASE(8, 2, 1) RDM_SPMM_CASE(8, 2, 2) RDM_SPMM_CASE(8, 2, 4)
    RDM_SPMM_CASE(8, 3, 1) RDM_SPMM_CASE(8, 3, 2) RDM_SPMM_CASE(8, 4, 1) RDM_SPMM_CASE(8, 4, 2)
    RDM_SPMM_CASE(16, 1, 1) RDM_SPMM_CASE(16, 1, 2) RDM_SPMM_CASE(16, 1, 4) RDM_SPMM_CASE(16, 2, 1)
    RDM_SPMM_CASE(16, 2, 2) RDM_SPMM_CASE(16, 2, 4) RDM_SPMM_CASE(16, 3, 1) RDM_SPMM_CASE(16, 3, 2)
    RDM_SPMM_CASE(16, 4, 1) RDM_SPMM_CASE(16, 4, 2) RDM_SPMM_CASE(32, 1, 1) RDM_SPMM_CASE(32, 1, 2)
    RDM_SPMM_CASE(32, 1, 4) RDM_SPMM_CASE(8, 1, 8)
    throw Error(RDM_ERR_ARG, "spmm: no kernel for G/V/U");
#undef RDM_SPMM_CASE
    if (conc) {
      RDM_CUDA(cudaEventRecord(ctx->aux_join, ctx->aux));
      RDM_CUDA(cudaStreamWaitEvent(ctx->stream, ctx->aux_join, 0));
    }
  }
heavy:
  if (A.n_heavy) {
    spmm_heavy_reduce<<<(unsigned)A.n_heavy, 128, 0, ctx->stream>>>(
        A.heavy_rows->as<int32_t>(), A.heavy_seg->as<int32_t>(), part, ldp, out, ld_out, w4, epi);
    RDM_LAUNCHED(ctx);
  }
}
}  // namespace

namespace {
__global__ void ref_count_kernel(const int32_t* __restrict__ col, int64_t nnz, int32_t* __restrict__ cnt) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nnz; j += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + col[j], 1);
}
__global__ void iota_kernel(int32_t* __restrict__ v, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    v[i] = (int32_t)i;
}
__global__ void hot_rank_kernel(const int32_t* __restrict__ order, int64_t hmax, int32_t* __restrict__ rank) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < hmax; i += (int64_t)gridDim.x * blockDim.x)
    rank[order[i]] = (int32_t)i;
}
__global__ void hot_encode_kernel(const int32_t* __restrict__ col, int64_t nnz, const int32_t* __restrict__ rank,
                                  int32_t* __restrict__ out) {
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nnz; j += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = col[j];
    const int32_t r = rank[c];
    out[j] = r;   // every column has a rank
  }
}
}  // namespace

// Column relabelling (see Hot) — an experiment, OFF by default: measured
// slower on the products-shaped graph (w = 256: 8.7 → 9.7 ms per call, the
// extra gather pass costs more than the locality gains) and ≈ 4 % faster on
// the papers100M-shaped one-rank SpMM (profiles/r2_relabel.md).
// RDM_RELABEL=1 at rdm_set_graph builds it for CSRs with >= 1 M input rows.
// Columns ranked by reference count (stable, descending); col_hot[j] = rank
// of col[j]; hot_ids = order.
void build_hot(rdm_ctx* ctx, Csr& A) {
  const char* on = getenv("RDM_RELABEL");
  const int64_t nin = A.in_rows();
  if (!(on && atoi(on)) || A.nnz == 0 || nin < (1 << 20) || nin >= INT32_MAX) return;
  const int64_t hmax = nin;   // every column ranked: the slice is gathered whole into rank order
  DevBuf cnt(nin * 4), iota(nin * 4), keys(nin * 4), order(nin * 4), rank(nin * 4);
  const unsigned g = (unsigned)(ctx->num_sms * 8);
  RDM_CUDA(cudaMemsetAsync(cnt.ptr, 0, nin * 4, ctx->stream));
  ref_count_kernel<<<g, 256, 0, ctx->stream>>>(A.col->as<int32_t>(), A.nnz, cnt.as<int32_t>());
  RDM_LAUNCHED(ctx);
  iota_kernel<<<g, 256, 0, ctx->stream>>>(iota.as<int32_t>(), nin);
  RDM_LAUNCHED(ctx);
  size_t tb = 0;
  RDM_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, cnt.as<int32_t>(), keys.as<int32_t>(),
                                                      iota.as<int32_t>(), order.as<int32_t>(), (int)nin, 0, 32,
                                                      ctx->stream));
  DevBuf tmp(std::max<size_t>(tb, 256));
  RDM_CUDA(cub::DeviceRadixSort::SortPairsDescending(tmp.ptr, tb, cnt.as<int32_t>(), keys.as<int32_t>(),
                                                      iota.as<int32_t>(), order.as<int32_t>(), (int)nin, 0, 32,
                                                      ctx->stream));
  RDM_CUDA(cudaMemsetAsync(rank.ptr, 0xFF, nin * 4, ctx->stream));   // -1 = cold
  hot_rank_kernel<<<g, 256, 0, ctx->stream>>>(order.as<int32_t>(), hmax, rank.as<int32_t>());
  RDM_LAUNCHED(ctx);
  A.col_hot.reset(new DevBuf(A.nnz * 4));
  hot_encode_kernel<<<g, 256, 0, ctx->stream>>>(A.col->as<int32_t>(), A.nnz, rank.as<int32_t>(),
                                                A.col_hot->as<int32_t>());
  RDM_LAUNCHED(ctx);
  A.hot_ids.reset(new DevBuf(hmax * 4));
  RDM_CUDA(cudaMemcpyAsync(A.hot_ids->ptr, order.ptr, hmax * 4, cudaMemcpyDeviceToDevice, ctx->stream));
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  A.hot_max = hmax;
}

// Row bins (host, one-time at rdm_set_graph; pure indexing of rowptr).
void build_bins(rdm_ctx* ctx, Csr& A, const int64_t* rp, bool sync) {
  const int64_t n = A.n;
  std::vector<int64_t> cnt(kSeg + 2, 0);
  int64_t n_heavy = 0, n_seg = 0, max_deg = 0;
  for (int64_t i = 0; i < n; ++i) {
    const int64_t d = rp[i + 1] - rp[i];
    max_deg = std::max(max_deg, d);
    if (d > kSeg) {
      ++n_heavy;
      n_seg += ceil_div(d, kSeg);
    } else {
      cnt[kSeg - d]++;  // descending degree
    }
  }
  const int64_t n_light = n - n_heavy;
  std::vector<int64_t> pos(kSeg + 2, 0);
  for (int64_t b = 1; b < kSeg + 2; ++b) pos[b] = pos[b - 1] + cnt[b - 1];
  // the bins are written straight into pinned staging, uploaded asynchronously:
  //   seg_start int64[n_seg] | seg_row int32[n_seg] | light int32[n_light] |
  //   heavy int32[n_heavy] | heavy_seg int32[n_heavy+1]
  const size_t b_seg = (size_t)n_seg * (sizeof(int64_t) + sizeof(int32_t));
  const size_t b_light = (size_t)n_light * sizeof(int32_t);
  const size_t b_heavy = (size_t)n_heavy * sizeof(int32_t);
  const size_t b_hseg = (size_t)(n_heavy + 1) * sizeof(int32_t);
  char* st = A.bins_stage.get<char>(b_seg + b_light + b_heavy + b_hseg + 64);
  int64_t* seg_start = reinterpret_cast<int64_t*>(st);
  int32_t* seg_row = reinterpret_cast<int32_t*>(st + (size_t)n_seg * sizeof(int64_t));
  int32_t* light = reinterpret_cast<int32_t*>(st + b_seg);
  int32_t* heavy = reinterpret_cast<int32_t*>(st + b_seg + b_light);
  int32_t* heavy_seg = reinterpret_cast<int32_t*>(st + b_seg + b_light + b_heavy);
  int64_t s = 0, h = 0;
  for (int64_t i = 0; i < n; ++i) {
    const int64_t d = rp[i + 1] - rp[i];
    if (d > kSeg) {
      heavy[h] = (int32_t)i;
      heavy_seg[h] = (int32_t)s;
      ++h;
      for (int64_t b = rp[i]; b < rp[i + 1]; b += kSeg) {
        seg_start[s] = b;
        seg_row[s] = (int32_t)i;
        ++s;
      }
    } else {
      light[pos[kSeg - d]++] = (int32_t)i;
    }
  }
  heavy_seg[n_heavy] = (int32_t)s;
  A.n_light = n_light;
  {
    // cnt[kSeg - d] = light rows of degree d
    int64_t acc = 0;
    for (int d = (int)kSeg; d >= 0; --d) {
      acc += cnt[kSeg - d];
      if (d <= Csr::kDegTab) A.deg_ge[d] = acc;
    }
  }
  A.n_seg = n_seg;
  A.n_heavy = n_heavy;
  A.max_deg = max_deg;
  // capacity is reused across calls (a GraphSAINT sampler rebuilds bins per subgraph)
  ensure_ws(A.light_rows, std::max<int64_t>(1, n_light) * sizeof(int32_t));
  // seg_start (int64) followed by seg_row (int32) in one allocation
  ensure_ws(A.seg_start, std::max<int64_t>(1, n_seg) * (sizeof(int64_t) + sizeof(int32_t)));
  ensure_ws(A.heavy_rows, std::max<int64_t>(1, n_heavy) * sizeof(int32_t));
  ensure_ws(A.heavy_seg, (n_heavy + 1) * sizeof(int32_t));
  const cudaMemcpyKind h2d = cudaMemcpyHostToDevice;
  if (n_light) RDM_CUDA(cudaMemcpyAsync(A.light_rows->ptr, light, b_light, h2d, ctx->stream));
  if (n_seg) RDM_CUDA(cudaMemcpyAsync(A.seg_start->ptr, seg_start, b_seg, h2d, ctx->stream));
  if (n_heavy) RDM_CUDA(cudaMemcpyAsync(A.heavy_rows->ptr, heavy, b_heavy, h2d, ctx->stream));
  RDM_CUDA(cudaMemcpyAsync(A.heavy_seg->ptr, heavy_seg, b_hseg, h2d, ctx->stream));
  if (sync) RDM_CUDA(cudaStreamSynchronize(ctx->stream));
}

// Dense hub core (one-time, host side, at rdm_set_graph for symmetric A):
// rank vertices by degree, take the K (multiple of 128) highest-degree ones
// whose mutual block pays for itself on the tensor cores (core_pays at the
// reference width 128), move A[hubs, hubs] into a dense K x K matrix and keep
// every other entry in a residual CSR.  K = 0 (no core) for graphs without a
// dense hub block.  Set RDM_NO_CORE=1 to disable.
void build_core(rdm_ctx* ctx, Csr& A, const int64_t* rp, const int32_t* col, const float* val) {
  (void)ctx;
  const int64_t n = A.n, nnz = A.nnz;
  const char* off = getenv("RDM_NO_CORE");
  if ((off && atoi(off)) || nnz == 0) return;
  if (build_hub_tiles(ctx, A, rp, col, val)) return;   // values factor: binary tiles
  if (n < 4096) return;
  std::vector<int32_t> order(n);
  for (int64_t i = 0; i < n; ++i) order[i] = (int32_t)i;
  std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
    return rp[a + 1] - rp[a] > rp[b + 1] - rp[b];
  });
  std::vector<int32_t> rank(n);
  for (int64_t i = 0; i < n; ++i) rank[order[i]] = (int32_t)i;
  const int64_t kmax = std::min<int64_t>((n / 2) / 128 * 128, 20480);
  if (kmax < 1024) return;
  std::vector<int64_t> hist(kmax + 1, 0);  // entries whose max(rank_r, rank_c) falls in bucket
  for (int64_t i = 0; i < n; ++i) {
    const int32_t ri = rank[i];
    for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
      const int32_t m = std::max(ri, rank[col[j]]);
      hist[m < kmax ? m : kmax]++;
    }
  }
  std::vector<int64_t> bucket(kmax / 128, 0);
  for (int64_t m = 0; m < kmax; ++m) bucket[m / 128] += hist[m];
  bool forced = false;
  const int64_t best_K = choose_core_K(bucket.data(), kmax, getenv("RDM_CORE_K"), &forced);
  if (!best_K) return;
  const int64_t K = best_K;
  A.core.forced = forced;
  std::vector<float> dense((size_t)K * K, 0.f);
  std::vector<int64_t> rrp(n + 1, 0);
  for (int64_t i = 0; i < n; ++i) {
    int64_t keep = 0;
    for (int64_t j = rp[i]; j < rp[i + 1]; ++j)
      keep += !(rank[i] < K && rank[col[j]] < K);
    rrp[i + 1] = rrp[i] + keep;
  }
  const int64_t rnnz = rrp[n];
  std::vector<int32_t> rcol(std::max<int64_t>(rnnz, 1));
  std::vector<float> rval(std::max<int64_t>(rnnz, 1));
  for (int64_t i = 0; i < n; ++i) {
    int64_t o = rrp[i];
    for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
      const int32_t c = col[j];
      if (rank[i] < K && rank[c] < K) {
        dense[(size_t)rank[i] * K + rank[c]] += val[j];
      } else {
        rcol[o] = c;
        rval[o] = val[j];
        ++o;
      }
    }
  }
  std::vector<int32_t> slot(n);
  for (int64_t v = 0; v < n; ++v) slot[v] = rank[v] < K ? rank[v] : -1;
  Core& c = A.core;
  c.K = K;
  c.nnz = nnz - rnnz;
  c.A.reset(new DevBuf((size_t)K * K * sizeof(float)));
  RDM_CUDA(cudaMemcpy(c.A->ptr, dense.data(), (size_t)K * K * sizeof(float), cudaMemcpyHostToDevice));
  c.hub_ids.reset(new DevBuf(K * sizeof(int32_t)));
  RDM_CUDA(cudaMemcpy(c.hub_ids->ptr, order.data(), K * sizeof(int32_t), cudaMemcpyHostToDevice));
  c.hub_slot.reset(new DevBuf(n * sizeof(int32_t)));
  RDM_CUDA(cudaMemcpy(c.hub_slot->ptr, slot.data(), n * sizeof(int32_t), cudaMemcpyHostToDevice));
  c.resid.reset(new Csr());
  Csr& R = *c.resid;
  R.n = n;
  R.nnz = rnnz;
  R.rowptr.reset(new DevBuf((n + 1) * sizeof(int64_t)));
  R.col.reset(new DevBuf(std::max<int64_t>(rnnz, 1) * sizeof(int32_t)));
  R.val.reset(new DevBuf(std::max<int64_t>(rnnz, 1) * sizeof(float)));
  RDM_CUDA(cudaMemcpy(R.rowptr->ptr, rrp.data(), (n + 1) * sizeof(int64_t), cudaMemcpyHostToDevice));
  if (rnnz) {
    RDM_CUDA(cudaMemcpy(R.col->ptr, rcol.data(), rnnz * sizeof(int32_t), cudaMemcpyHostToDevice));
    RDM_CUDA(cudaMemcpy(R.val->ptr, rval.data(), rnnz * sizeof(float), cudaMemcpyHostToDevice));
  }
  build_bins(ctx, R, rrp.data());
}

}  // namespace rdm
