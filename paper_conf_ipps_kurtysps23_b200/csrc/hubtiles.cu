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
// * b is exact in bf16 → the A operand of a kind::f16 MMA is exact; tiles are
//   stored as bits (2 KB per 128 x 128 tile, vs 64 KB fp32) and expanded to
//   bf16 in shared memory;
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
//   warp 0 TMA producer: per 64-wide k stage the tile half's bits (1 KB, bulk
//          copy) and the three B pieces (n_mma x 64 bf16 each, 128B swizzle)
//   warp 1 MMA issuer: 4 k16 steps x 3 pieces of tcgen05.mma kind::f16 per
//          stage into a double-buffered TMEM accumulator (128 x n_mma fp32)
//   warp 2 TMEM allocator
//   warps 4-7 expander: bits → 0/1 bf16 A half-tile (128 x 64, swizzled smem)
//   warps 8-11 epilogue: tcgen05.ld → partial rows of the work item → global
// A work item is a run of ≤ `chunk` tiles of one 128-row block; its 128 x w
// partial goes to part[item] and the SpMM epilogue sums the items of the row's
// block in item order.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>
#include <cuda_fp16.h>

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
// the same with A/B fp16 (format 0)
__host__ __device__ constexpr uint32_t idesc_f16(int N) {
  return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

__device__ __forceinline__ void bulk_load(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"((uint64_t)src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void tma_load_4d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1,
                                            int c2, int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(
          smem_u32(dst)),
      "l"((uint64_t)map), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
      : "memory");
}

// kind::f16 MMA with A from TMEM (bf16 pairs packed in 32-bit columns).
__device__ __forceinline__ void tc_mma_f16_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t idesc,
                                              uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void tmem_st32u(uint32_t addr, const uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,"
      "%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(addr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]),
      "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]),
      "r"(v[16]), "r"(v[17]), "r"(v[18]), "r"(v[19]), "r"(v[20]), "r"(v[21]), "r"(v[22]), "r"(v[23]),
      "r"(v[24]), "r"(v[25]), "r"(v[26]), "r"(v[27]), "r"(v[28]), "r"(v[29]), "r"(v[30]), "r"(v[31])
      : "memory");
}

// explicit shared-memory loads (the aligned dynamic-smem pointer is generic to
// the compiler, which otherwise emits generic LD for the expander's hot loop)
__device__ __forceinline__ uint4 lds128(uint32_t addr) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(addr));
  return v;
}
__device__ __forceinline__ uint2 lds64(uint32_t addr) {
  uint2 v;
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(addr) : "memory");
  return v;
}

// Two bits → two bf16 (0 or 1.0 = 0x3F80) packed in one 32-bit word.
__device__ __forceinline__ uint32_t bits2_bf16(uint32_t b) {
  return ((b & 1u) * 0x3F80u) | (((b >> 1) & 1u) * 0x3F800000u);
}
// … or two fp16 (1.0 = 0x3C00).
__device__ __forceinline__ uint32_t bits2_f16(uint32_t b) {
  return ((b & 1u) * 0x3C00u) | (((b >> 1) & 1u) * 0x3C000000u);
}

// Launch shape of one product (host-computed).
struct TileShape {
  int n_items, tiles_n, n_mma;
  int64_t w, ldp;
  int S, SA;          // shared-memory stages, TMEM A slots
  int HS;             // 64-wide k halves per stage (1 or 2)
  int stage_bytes;    // HS · (NP · n_mma · 128 + 1024)
  int R;              // > 0: concatenated-piece MMAs with R rotating accumulator sets
  int acc_cols;       // TMEM columns per accumulator buffer
  int dbg;            // timing experiments (RDM_TILE_DBG): 1 = skip the MMAs, 2 = the i8 expansion, 4 = the i8 stores
  const float* colscale;   // NP == 2: 2^e_n per output column (fp16 pieces are column-scaled)
};

// NP = pieces of s⊙X: 2 fp16 pieces with a per-column power-of-two scale
// (22 significant bits, fp32-class: RDM_PREC_FP32), 3 bf16 pieces (24 bits,
// kept for comparison: RDM_TILE_PIECES=3) or 1 bf16 piece (RDM_PREC_FAST).
template <int HS, int NP>
__global__ void __launch_bounds__(384, 1)
hub_tile_kernel(const __grid_constant__ CUtensorMap tmB, const __grid_constant__ CUtensorMap tmB2d,
                const uint64_t* __restrict__ bits,
                const int32_t* __restrict__ tile_cb, const int32_t* __restrict__ item_tb,
                float* __restrict__ part, const TileShape sh) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int S = sh.S, SA = sh.SA, R = sh.R, n_mma = sh.n_mma;
  uint64_t* full = (uint64_t*)(smem + S * sh.stage_bytes);
  uint64_t* empty = full + S;
  uint64_t* conv = empty + S;    // [SA] TMEM A slot expanded
  uint64_t* aempty = conv + SA;  // [SA] TMEM A slot consumed by its MMAs
  uint64_t* tfull = aempty + SA; // [2]
  uint64_t* tempty = tfull + 2;  // [2]
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  uint4* lut = (uint4*)(smem + S * sh.stage_bytes + 1024);   // byte → 8 bf16 (0 / 1)
  const uint32_t lut_s = smem_u32(lut);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int total = sh.n_items * sh.tiles_n;
  for (int i = threadIdx.x; i < 256; i += blockDim.x)
    lut[i] = NP == 2 ? make_uint4(bits2_f16(i), bits2_f16(i >> 2), bits2_f16(i >> 4), bits2_f16(i >> 6))
                     : make_uint4(bits2_bf16(i), bits2_bf16(i >> 2), bits2_bf16(i >> 4), bits2_bf16(i >> 6));
  // Two rings.  Shared-memory stage s: the B pieces of HS k-halves as
  // [half][piece][n_mma][64 bf16] (one 4-D TMA; pieces of a half adjacent, so
  // a concatenated MMA of N = 3 n_mma reads all three), then the halves' bits
  // [half][128 rows] u64.  TMEM: two accumulator buffers of acc_cols columns,
  // then SA A slots of 32·HS columns (64·HS bf16 per row, packed in pairs).
  const int bpiece = n_mma * 128;                 // bytes of one piece of one half
  const int bbytes = HS * NP * bpiece;
  const uint32_t kAcol = 2 * sh.acc_cols;
  auto B_st = [&](int s) { return smem + s * sh.stage_bytes; };
  auto bits_st = [&](int s) { return smem + s * sh.stage_bytes + bbytes; };

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < SA; ++i) {
      mbar_init(&conv[i], 128);
      mbar_init(&aempty[i], 1);
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
                 "n"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const int spt = (TK / SK) / HS;                 // stages per tile

  // Every role walks the same stage sequence with (slot, phase) counters (no
  // divisions on the single-thread issue paths).
  if (warp == 0) {
    if (lane == 0) {
      int s = 0;
      uint32_t ph = 0, kc = 0;
      const uint32_t bytes = (uint32_t)bbytes + HS * 1024;
      for (int t = blockIdx.x; t < total; t += gridDim.x) {
        const int item = t / sh.tiles_n;
        const int n0 = (t % sh.tiles_n) * 128;
        const int tb = item_tb[item], T = item_tb[item + 1] - tb;
        // items start at a per-item rotation of their tile run, so that the
        // CTAs working on neighbouring row blocks (whose tiles share column
        // blocks) do not all read the same B panel lines at once
        int ti = (int)(((unsigned)item * 2654435761u) % (unsigned)max(T, 1));
        for (int i = 0; i < T; ++i) {
          const int tile = tb + ti;
          if (++ti == T) ti = 0;
          const int kb = tile_cb[tile] * (TK / SK);   // first 64-wide k block of the tile
          for (int h = 0; h < spt; ++h) {
            if (kc >= (uint32_t)S) mbar_wait(&empty[s], ph ^ 1);
            mbar_expect_tx(&full[s], bytes);
            bulk_load(bits_st(s), bits + ((int64_t)tile * 2 + h * HS) * TK, HS * 1024, &full[s]);
            if (HS == 2) {
              tma_load_4d(B_st(s), &tmB, &full[s], 0, n0, 0, kb);
            } else {   // three 2-D boxes from the stacked panels (measured faster for one half)
              for (int pc = 0; pc < NP; ++pc)
                tma_load_2d(B_st(s) + pc * bpiece, &tmB2d, &full[s], (kb + h) * SK, pc * (int)sh.w + n0);
            }
            ++kc;
            if (++s == S) { s = 0; ph ^= 1; }
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      const uint32_t idesc = NP == 2 ? idesc_f16(R ? NP * n_mma : n_mma) : idesc_bf16(R ? NP * n_mma : n_mma);
      // descriptors advance linearly: +stage_bytes per stage, +3·bpiece per
      // k half, +bpiece per piece, +32 B per k16 step (16-byte units)
      const uint64_t bd0 = sdesc(smem_u32(B_st(0)), 16, 1024);
      const uint32_t st16 = (uint32_t)sh.stage_bytes >> 4, pc16 = (uint32_t)bpiece >> 4;
      const uint32_t rho_step = (uint32_t)NP * n_mma, rho_end = (uint32_t)R * rho_step;
      int s = 0, a = 0;
      uint32_t ph = 0, aph = 0;
      int it = 0;
      for (int t = blockIdx.x; t < total; t += gridDim.x, ++it) {
        const int item = t / sh.tiles_n;
        const int nst = (item_tb[item + 1] - item_tb[item]) * spt;
        const int acc = it & 1;
        if (it >= 2) mbar_wait(&tempty[acc], ((it >> 1) - 1) & 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * sh.acc_cols;
        uint32_t rho = 0;      // rotating accumulator set offset (R > 0)
        int g = 0;             // k16 steps issued for this item
        for (int st = 0; st < nst; ++st) {
          mbar_wait(&conv[a], aph);
          tc_fence_after();
          const uint32_t ta = tmem_base + kAcol + a * 32 * HS;
          const uint64_t bd = bd0 + (uint64_t)(s * st16);
          if (!(sh.dbg & 1)) {
#pragma unroll
            for (int h = 0; h < HS; ++h) {
              const uint64_t bh = bd + (uint64_t)(h * NP * pc16);
              const uint32_t th = ta + h * 32;
              if (R) {
#pragma unroll
                for (int j = 0; j < SK / 16; ++j, ++g) {
                  tc_mma_f16_ts(d_tmem + rho, th + j * 8, bh + 2 * j, idesc, g >= R ? 1u : 0u);
                  rho += rho_step;
                  if (rho == rho_end) rho = 0;
                }
              } else {
#pragma unroll
                for (int j = 0; j < SK / 16; ++j, ++g) {   // 8 packed A columns, 32 B of B rows per k16
                  tc_mma_f16_ts(d_tmem, th + j * 8, bh + 2 * j, idesc, g > 0 ? 1u : 0u);
#pragma unroll
                  for (int pc = 1; pc < NP; ++pc)
                    tc_mma_f16_ts(d_tmem, th + j * 8, bh + pc * pc16 + 2 * j, idesc, 1u);
                }
              }
            }
          }
          tc_commit(&empty[s]);
          tc_commit(&aempty[a]);
          if (++s == S) { s = 0; ph ^= 1; }
          if (++a == SA) { a = 0; aph ^= 1; }
        }
        tc_commit(&tfull[acc]);
      }
    }
  } else if (warp >= 4 && warp < 8) {
    // expander: row r of the stage's A tile part from its bits → bf16 0 / 1
    // (one table lookup per byte), two per 32-bit TMEM column, stored to TMEM
    // lane r (the warp's lane quadrant): the MMAs read A from TMEM.
    const int r = threadIdx.x - 128;
    const uint32_t lane_off = (uint32_t)((warp & 3) * 32) << 16;
    int s = 0, a = 0;
    uint32_t ph = 0, aph = 0, kc = 0;
    for (int t = blockIdx.x; t < total; t += gridDim.x) {
      const int item = t / sh.tiles_n;
      const int nst = (item_tb[item + 1] - item_tb[item]) * spt;
      for (int st = 0; st < nst; ++st, ++kc) {
        mbar_wait(&full[s], ph);
        if (kc >= (uint32_t)SA) {
          mbar_wait(&aempty[a], aph ^ 1);
          tc_fence_after();
        }
#pragma unroll
        for (int h = 0; h < HS; ++h) {
          const uint2 b = lds64(smem_u32(bits_st(s) + h * 1024) + r * 8);
          uint32_t v[32];
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const uint4 e = lds128(lut_s + (((i < 4 ? b.x : b.y) >> (8 * (i & 3))) & 0xFFu) * 16);
            v[4 * i] = e.x; v[4 * i + 1] = e.y; v[4 * i + 2] = e.z; v[4 * i + 3] = e.w;
          }
          tmem_st32u(tmem_base + lane_off + kAcol + a * 32 * HS + h * 32, v);
        }
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        tc_fence_before();
        mbar_arrive(&conv[a]);
        if (++s == S) { s = 0; ph ^= 1; }
        if (++a == SA) { a = 0; aph ^= 1; }
      }
    }
  } else if (warp >= 8) {
    const int q = warp & 3;
    int it = 0;
    for (int t = blockIdx.x; t < total; t += gridDim.x, ++it) {
      const int item = t / sh.tiles_n;
      const int64_t n0 = (int64_t)(t % sh.tiles_n) * 128;
      const int acc = it & 1;
      mbar_wait_sleep(&tfull[acc], (it >> 1) & 1);
      tc_fence_after();
      float* prow = part + ((int64_t)item * TK + q * 32 + lane) * sh.ldp + n0;
      for (int c0 = 0; c0 < n_mma; c0 += 32) {
        if (n0 + c0 >= sh.w) break;
        uint32_t rr[32];
        const uint32_t a0 = tmem_base + acc * sh.acc_cols + ((uint32_t)(q * 32) << 16) + (uint32_t)c0;
        if (R) {   // fixed order: lo, mid, hi pieces, each over its rotations
          float sum[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) sum[i] = 0.f;
          for (int pc = NP - 1; pc >= 0; --pc)
            for (int rho = 0; rho < R; ++rho) {
              tmem_ld32(a0 + (uint32_t)((rho * NP + pc) * n_mma), rr);
#pragma unroll
              for (int i = 0; i < 32; ++i) sum[i] += __uint_as_float(rr[i]);
            }
#pragma unroll
          for (int i = 0; i < 32; ++i) rr[i] = __float_as_uint(sum[i]);
        } else {
          tmem_ld32(a0, rr);
        }
#pragma unroll
        for (int i = 0; i < 32; i += 4)
          if (n0 + c0 + i < sh.w) {
            float4 o = make_float4(__uint_as_float(rr[i]), __uint_as_float(rr[i + 1]), __uint_as_float(rr[i + 2]),
                                   __uint_as_float(rr[i + 3]));
            if (NP == 2) {   // undo the column scale of the fp16 pieces (exact: powers of two)
              const float4 cs = __ldg(reinterpret_cast<const float4*>(sh.colscale + n0 + c0 + i));
              o.x *= cs.x; o.y *= cs.y; o.z *= cs.z; o.w *= cs.w;
            }
            *reinterpret_cast<float4*>(prow + c0 + i) = o;
          }
      }
      tc_fence_before();
      mbar_arrive(&tempty[acc]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(512));
  }
}

// B pieces: P_p[n][k] = piece p of s_k · X[hub_k][n] (K-major rows of length K2),
// transposed through shared memory.  hi = bf16(x), mid = bf16(x − hi),
// lo = bf16(x − hi − mid); the differences are exact in fp32.
__global__ void tile_panels_kernel(const float* __restrict__ X, int64_t ldx, const int32_t* __restrict__ hub_ids,
                                   const float* __restrict__ scale, int64_t K2, int64_t w,
                                   __nv_bfloat16* __restrict__ p0, __nv_bfloat16* __restrict__ p1,
                                   __nv_bfloat16* __restrict__ p2, int np) {
  __shared__ float t[64][33];
  const int64_t k0 = (int64_t)blockIdx.x * 64, n0 = (int64_t)blockIdx.y * 32;
  {
    // the 8 hub ids first, then 8 independent row gathers per thread
    const int64_t n = n0 + threadIdx.x;
    int32_t id[8];
    float sc[8], x[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      id[u] = __ldg(hub_ids + k0 + threadIdx.y + 8 * u);
      sc[u] = __ldg(scale + k0 + threadIdx.y + 8 * u);
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) x[u] = (n < w) ? __ldg(X + (int64_t)id[u] * ldx + n) : 0.f;
#pragma unroll
    for (int u = 0; u < 8; ++u) t[threadIdx.y + 8 * u][threadIdx.x] = sc[u] * x[u];
  }
  __syncthreads();
  for (int i = threadIdx.y; i < 32; i += 8) {
    const int64_t n = n0 + i;
    if (n >= w) break;
    // a pair of consecutive k per thread: 4-byte stores, 128 B per warp and piece
    const int kk = 2 * threadIdx.x;
    const float x0 = t[kk][i], x1 = t[kk + 1][i];
    const __nv_bfloat162 h = __floats2bfloat162_rn(x0, x1);
    const float r0 = x0 - __low2float(h), r1 = x1 - __high2float(h);
    const __nv_bfloat162 m = __floats2bfloat162_rn(r0, r1);
    const __nv_bfloat162 l = __floats2bfloat162_rn(r0 - __low2float(m), r1 - __high2float(m));
    const int64_t o = n * K2 + k0 + kk;
    *reinterpret_cast<__nv_bfloat162*>(p0 + o) = h;
    if (np == 3) {
      *reinterpret_cast<__nv_bfloat162*>(p1 + o) = m;
      *reinterpret_cast<__nv_bfloat162*>(p2 + o) = l;
    }
  }
}

// Column maxima of |s_k · X[hub_k][n]| over the K2 hub slots (bit patterns of
// non-negative floats order like unsigned ints: atomicMax is exact and
// order-independent).  Block: 32 columns x 8 k-lanes, 32 k per lane (short
// dependent gather chains: the hub id, then the row).
__global__ void tile_colmax_kernel(const float* __restrict__ X, int64_t ldx, const int32_t* __restrict__ hub_ids,
                                   const float* __restrict__ scale, int64_t K2, int64_t w,
                                   unsigned int* __restrict__ colmax) {
  __shared__ float red[8][33];
  const int64_t n = (int64_t)blockIdx.y * 32 + threadIdx.x;
  const int64_t k0 = (int64_t)blockIdx.x * 256;
  float m = 0.f;
  if (n < w) {
    // K2 is a multiple of 128 and blocks start at multiples of 256: a block's
    // k range is full or half full; batches of 8 independent gathers per thread
    const int64_t k1 = min(K2, k0 + 256);
    for (int64_t kb = k0 + threadIdx.y; kb < k1; kb += 64) {
      int32_t id[8];
      float sc[8], x[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        id[u] = __ldg(hub_ids + kb + 8 * u);
        sc[u] = __ldg(scale + kb + 8 * u);
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) x[u] = __ldg(X + (int64_t)id[u] * ldx + n);
#pragma unroll
      for (int u = 0; u < 8; ++u) m = fmaxf(m, fabsf(sc[u] * x[u]));
    }
  }
  red[threadIdx.y][threadIdx.x] = m;
  __syncthreads();
  if (threadIdx.y == 0 && n < w) {
    for (int i = 1; i < 8; ++i) m = fmaxf(m, red[i][threadIdx.x]);
    atomicMax(colmax + n, __float_as_uint(m));
  }
}

// fp16 pieces: y = s_k · X[hub_k][n] · 2^-e_n with e_n chosen so that the
// column maximum lands in [2^13, 2^14) (far from fp16 overflow), hi = fp16(y),
// lo = fp16(y − hi) (the difference is exact in fp32): 22 significant bits.
// colscale[n] = 2^e_n for the epilogue.
__global__ void tile_panels_f16_kernel(const float* __restrict__ X, int64_t ldx, const int32_t* __restrict__ hub_ids,
                                       const float* __restrict__ scale, int64_t K2, int64_t w,
                                       const unsigned int* __restrict__ colmax, __half* __restrict__ p0,
                                       __half* __restrict__ p1, float* __restrict__ colscale) {
  __shared__ float t[64][33];
  __shared__ float inv[32];
  const int64_t k0 = (int64_t)blockIdx.x * 64, n0 = (int64_t)blockIdx.y * 32;
  if (threadIdx.y == 0) {
    const int64_t n = n0 + threadIdx.x;
    const float mx = n < w ? __uint_as_float(colmax[n]) : 0.f;
    const int e = mx > 0.f ? ilogbf(mx) - 13 : 0;
    inv[threadIdx.x] = ldexpf(1.f, -e);
    if (blockIdx.x == 0 && n < w) colscale[n] = ldexpf(1.f, e);
  }
  {
    // the 8 hub ids first, then 8 independent row gathers per thread
    const int64_t n = n0 + threadIdx.x;
    int32_t id[8];
    float sc[8], x[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      id[u] = __ldg(hub_ids + k0 + threadIdx.y + 8 * u);
      sc[u] = __ldg(scale + k0 + threadIdx.y + 8 * u);
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) x[u] = (n < w) ? __ldg(X + (int64_t)id[u] * ldx + n) : 0.f;
#pragma unroll
    for (int u = 0; u < 8; ++u) t[threadIdx.y + 8 * u][threadIdx.x] = sc[u] * x[u];
  }
  __syncthreads();
  for (int i = threadIdx.y; i < 32; i += 8) {
    const int64_t n = n0 + i;
    if (n >= w) break;
    const int kk = 2 * threadIdx.x;   // a pair of consecutive k per thread (4-byte stores)
    const float y0 = t[kk][i] * inv[i], y1 = t[kk + 1][i] * inv[i];
    const __half2 h = __floats2half2_rn(y0, y1);
    const __half2 l = __floats2half2_rn(y0 - __low2float(h), y1 - __high2float(h));
    const int64_t o = n * K2 + k0 + kk;
    *reinterpret_cast<__half2*>(p0 + o) = h;
    *reinterpret_cast<__half2*>(p1 + o) = l;
  }
}

// ---------------------------------------------------------------- int8 tiles
// kind::i8 form (default for fp32).  y = s_k · X[hub_k][n] · 2^-e_n with the
// column maximum scaled into [2^21, 2^22) is rounded to an integer v
// (|v| ≤ 2^22: 23 significant bits relative to the column maximum) and split
// into three signed 8-bit digits v = d2·2^16 + d1·2^8 + d0 (d ∈ [-128, 127]).
// The 0/1 tile is exact in int8, the MMAs accumulate in s32 exactly, so each
// output is Σ_j b_ij v_j computed exactly and rounded to fp32 once, ×2^e_n.
// Against the fp16 pair: the bit expansion is 2 integer ops per 4 elements
// (the nibble times 0x204081 spreads 4 bits over 4 bytes) instead of a table
// lookup per 8 bf16, the A operand is half the TMEM bytes, and the int8 MMA
// rate is twice the fp16 one (3 digits cost 1.5 fp16 MMAs, the pair 2).
constexpr int I8_NMAX = 64;                 // output columns per pass (3 digits → N ≤ 192)

__host__ __device__ constexpr uint32_t idesc_i8(int N) {
  // D s32 (2), A / B signed 8-bit (1), K-major both, M = 128
  return (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

__device__ __forceinline__ void tc_mma_i8_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t idesc,
                                             uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate)
      : "memory");
}

// One stage = TP whole tiles of one item: TP digit panels [D][n_mma][128 B]
// (128-byte swizzle, one 4-D TMA each), then the TP tiles' bits [half][128
// rows] u64; an item's last stage is padded with the all-zero tile.  TP = 2
// halves the per-stage handshakes (expander → MMA issuer → commits → ring
// slots): 355 → 318 µs per Reddit-shaped w = 128 call, 174 → 159 µs at w = 41
// (profiles/r2_tile_stages.md — halving the panel bytes alone changed nothing).
template <int D, int TP>
__global__ void __launch_bounds__(384, 1)
hub_tile_i8_kernel(const __grid_constant__ CUtensorMap tmB, const uint64_t* __restrict__ bits,
                   const uint64_t* __restrict__ zero_bits,
                   const int32_t* __restrict__ tile_cb, const int32_t* __restrict__ item_tb,
                   float* __restrict__ part, const TileShape sh) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int S = sh.S, SA = sh.SA, n_mma = sh.n_mma;
  uint64_t* full = (uint64_t*)(smem + S * sh.stage_bytes);
  uint64_t* empty = full + S;
  uint64_t* conv = empty + S;
  uint64_t* aempty = conv + SA;
  uint64_t* tfull = aempty + SA;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int total = sh.n_items * sh.tiles_n;
  const int bbytes = D * n_mma * 128;
  auto B_st = [&](int s, int u) { return smem + s * sh.stage_bytes + u * bbytes; };
  auto bits_st = [&](int s, int u) { return smem + s * sh.stage_bytes + TP * bbytes + u * 2048; };
  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < SA; ++i) {
      mbar_init(&conv[i], 128);
      mbar_init(&aempty[i], 1);
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
                 "n"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const uint32_t kAcol = 2 * sh.acc_cols;

  if (warp == 0) {
    // the whole warp fetches the column blocks of 32 tiles at a time (one
    // coalesced load instead of one dependent L2 round trip per tile on the
    // issue path); lane 0 issues the copies
    int s = 0;
    uint32_t ph = 0, kc = 0;
    // (timing experiments: 8 = load half of each digit panel, as one CTA of a
    // pair would; 16 = skip the bits copies)
    const uint32_t bytes =
        (uint32_t)TP * ((uint32_t)((sh.dbg & 8) ? bbytes / 2 : bbytes) + ((sh.dbg & 16) ? 0 : 2048));
    int u = 0;   // tile slot within the current stage
    for (int t = blockIdx.x; t < total; t += gridDim.x) {
      const int item = t / sh.tiles_n;
      const int n0 = (t % sh.tiles_n) * n_mma;
      const int tb = item_tb[item], T = item_tb[item + 1] - tb;
      const int rot = (int)(((unsigned)item * 2654435761u) % (unsigned)max(T, 1));
      const int Tp = (T + TP - 1) / TP * TP;   // padded with zero tiles
      for (int i0 = 0; i0 < Tp; i0 += 32) {
        int idx = rot + i0 + lane;
        idx -= (idx >= T) ? T : 0;
        idx -= (idx >= T) ? T : 0;
        const bool real = i0 + lane < T;
        const int my_tile = real ? tb + idx : -1;
        const int my_cb = real ? __ldg(tile_cb + tb + idx) : 0;
        const int cnt = min(32, Tp - i0);
        int last_cb = __shfl_sync(0xffffffffu, my_cb, 0);
        for (int k = 0; k < cnt; ++k) {
          const int tile = __shfl_sync(0xffffffffu, my_tile, k);
          int cb = __shfl_sync(0xffffffffu, my_cb, k);
          if (tile < 0) cb = last_cb;   // zero tile: any panel
          last_cb = cb;
          if (lane == 0) {
            if (u == 0) {
              if (kc >= (uint32_t)S) mbar_wait(&empty[s], ph ^ 1);
              mbar_expect_tx(&full[s], bytes);
            }
            if (!(sh.dbg & 16))
              bulk_load(bits_st(s, u), tile >= 0 ? bits + (int64_t)tile * 2 * TK : zero_bits, 2048, &full[s]);
            tma_load_4d(B_st(s, u), &tmB, &full[s], 0, n0, 0, cb);
          }
          if (++u == TP) {
            u = 0;
            ++kc;
            if (++s == S) { s = 0; ph ^= 1; }
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      const uint32_t idesc = idesc_i8(D * n_mma);
      const uint64_t bd0 = sdesc(smem_u32(B_st(0, 0)), 16, 1024);
      const uint32_t st16 = (uint32_t)sh.stage_bytes >> 4, bb16 = (uint32_t)bbytes >> 4;
      int s = 0, a = 0;
      uint32_t ph = 0, aph = 0;
      int it = 0;
      for (int t = blockIdx.x; t < total; t += gridDim.x, ++it) {
        const int item = t / sh.tiles_n;
        const int nst = (item_tb[item + 1] - item_tb[item] + TP - 1) / TP;
        const int acc = it & 1;
        if (it >= 2) mbar_wait(&tempty[acc], ((it >> 1) - 1) & 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * sh.acc_cols;
        for (int st = 0; st < nst; ++st) {
          mbar_wait(&conv[a], aph);
          tc_fence_after();
          if (!(sh.dbg & 1)) {
#pragma unroll
            for (int uu = 0; uu < TP; ++uu) {
              const uint32_t ta = tmem_base + kAcol + (a * TP + uu) * 32;
              const uint64_t bd = bd0 + (uint64_t)(s * st16 + uu * bb16);
#pragma unroll
              for (int j = 0; j < TK / 32; ++j)   // K = 32 int8 per MMA: 8 A columns, 32 B of B rows
                tc_mma_i8_ts(d_tmem, ta + j * 8, bd + 2 * j, idesc, (st | uu | j) ? 1u : 0u);
            }
          }
          tc_commit(&empty[s]);
          tc_commit(&aempty[a]);
          if (++s == S) { s = 0; ph ^= 1; }
          if (++a == SA) { a = 0; aph ^= 1; }
        }
        tc_commit(&tfull[acc]);
      }
    }
  } else if (warp >= 4 && warp < 8) {
    // expander: row r's 128 bits → 128 int8 0 / 1, four per 32-bit TMEM column
    const int r = threadIdx.x - 128;
    const uint32_t lane_off = (uint32_t)((warp & 3) * 32) << 16;
    int s = 0, a = 0;
    uint32_t ph = 0, aph = 0, kc = 0;
    for (int t = blockIdx.x; t < total; t += gridDim.x) {
      const int item = t / sh.tiles_n;
      const int nst = (item_tb[item + 1] - item_tb[item] + TP - 1) / TP;
      for (int st = 0; st < nst; ++st, ++kc) {
        mbar_wait(&full[s], ph);
        if (kc >= (uint32_t)SA) {
          mbar_wait(&aempty[a], aph ^ 1);
          tc_fence_after();
        }
        if (!(sh.dbg & 2)) {   // (timing experiments: 2 = skip the expansion)
#pragma unroll
          for (int uu = 0; uu < TP; ++uu) {
            const uint32_t bs = smem_u32(bits_st(s, uu)) + r * 8;
            const uint2 h0 = lds64(bs), h1 = lds64(bs + 1024);
            const uint32_t w4[4] = {h0.x, h0.y, h1.x, h1.y};
            uint32_t v[32];
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = (((w4[i >> 3] >> (4 * (i & 7))) & 15u) * 0x204081u) & 0x01010101u;
            tmem_st32u(tmem_base + lane_off + kAcol + (a * TP + uu) * 32, v);
          }
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        }
        tc_fence_before();
        mbar_arrive(&conv[a]);
        if (++s == S) { s = 0; ph ^= 1; }
        if (++a == SA) { a = 0; aph ^= 1; }
      }
    }
  } else if (warp >= 8) {
    const int q = warp & 3;
    int it = 0;
    for (int t = blockIdx.x; t < total; t += gridDim.x, ++it) {
      const int item = t / sh.tiles_n;
      const int64_t n0 = (int64_t)(t % sh.tiles_n) * n_mma;
      const int acc = it & 1;
      mbar_wait_sleep(&tfull[acc], (it >> 1) & 1);
      tc_fence_after();
      float* prow = part + ((int64_t)item * TK + q * 32 + lane) * sh.ldp + n0;
      for (int c0 = 0; c0 < n_mma; c0 += 32) {
        if (n0 + c0 >= sh.w) break;
        // digit accumulators, most significant first: v = Σ_d acc_d · 256^(D-1-d)
        uint32_t dg[D][32];
        const uint32_t a0 = tmem_base + acc * sh.acc_cols + ((uint32_t)(q * 32) << 16) + (uint32_t)c0;
#pragma unroll
        for (int d = 0; d < D; ++d) tmem_ld32(a0 + (uint32_t)(d * n_mma), dg[d]);
#pragma unroll
        for (int i = 0; i < 32; i += 4)
          if (n0 + c0 + i < sh.w && !(sh.dbg & 4)) {   // (4 = skip the stores)
            const float4 cs = __ldg(reinterpret_cast<const float4*>(sh.colscale + n0 + c0 + i));
            float o[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
              long long v = 0;
#pragma unroll
              for (int d = 0; d < D; ++d) v = v * 256 + (long long)(int)dg[d][i + u];
              o[u] = __ll2float_rn(v);
            }
            *reinterpret_cast<float4*>(prow + c0 + i) = make_float4(o[0] * cs.x, o[1] * cs.y, o[2] * cs.z, o[3] * cs.w);
          }
      }
      tc_fence_before();
      mbar_arrive(&tempty[acc]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(512));
  }
}

// Pair form of hub_tile_i8_kernel: a work unit is a run of merged entries
// of a row-block PAIR (2p, 2p+1); each stage carries ONE digit-panel load for
// the column block and both tiles' bits (a zero tile where a row block has
// none), and the MMA issuer multiplies both A tiles against it into two
// accumulators — half the panel ingress per tile.  TMEM: the two accumulators
// (single-buffered: 2·D·n_mma columns) then SA slots of 64 columns (the two
// expanded A tiles).  part holds 256 rows per item (rows 0-127: block 2p).
template <int D>
__global__ void __launch_bounds__(384, 1)
hub_tile_i8_pair_kernel(const __grid_constant__ CUtensorMap tmB, const uint64_t* __restrict__ bits,
                        const uint64_t* __restrict__ zero_bits, const int32_t* __restrict__ pm_cb,
                        const int32_t* __restrict__ pm_t1, const int32_t* __restrict__ pm_t2,
                        const int32_t* __restrict__ pitem_pm, float* __restrict__ part, const TileShape sh) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int S = sh.S, SA = sh.SA, n_mma = sh.n_mma;
  uint64_t* full = (uint64_t*)(smem + S * sh.stage_bytes);
  uint64_t* empty = full + S;
  uint64_t* conv = empty + S;
  uint64_t* aempty = conv + SA;
  uint64_t* tfull = aempty + SA;
  uint64_t* tempty = tfull + 1;
  uint32_t* tmem_slot = (uint32_t*)(tempty + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int total = sh.n_items * sh.tiles_n;
  const int bbytes = D * n_mma * 128;
  const int accw = D * n_mma;                      // columns of one accumulator
  auto B_st = [&](int s) { return smem + s * sh.stage_bytes; };
  auto bits_st = [&](int s) { return smem + s * sh.stage_bytes + bbytes; };   // [tile 2][half 2][128] u64
  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < SA; ++i) {
      mbar_init(&conv[i], 128);
      mbar_init(&aempty[i], 1);
    }
    mbar_init(&tfull[0], 1);
    mbar_init(&tempty[0], 128);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "n"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  const uint32_t kAcol = (uint32_t)sh.acc_cols;     // both accumulators, rounded up

  if (warp == 0) {
    int s = 0;
    uint32_t ph = 0, kc = 0;
    const uint32_t bytes = (uint32_t)bbytes + 4096;
    for (int t = blockIdx.x; t < total; t += gridDim.x) {
      const int item = t / sh.tiles_n;
      const int n0 = (t % sh.tiles_n) * n_mma;
      const int mb = pitem_pm[item], M = pitem_pm[item + 1] - mb;
      const int rot = (int)(((unsigned)item * 2654435761u) % (unsigned)max(M, 1));
      for (int i0 = 0; i0 < M; i0 += 32) {
        int idx = rot + i0 + lane;
        idx -= (idx >= M) ? M : 0;
        idx -= (idx >= M) ? M : 0;
        const bool ok = i0 + lane < M;
        const int my_cb = ok ? __ldg(pm_cb + mb + idx) : 0;
        const int my_t1 = ok ? __ldg(pm_t1 + mb + idx) : -1;
        const int my_t2 = ok ? __ldg(pm_t2 + mb + idx) : -1;
        const int cnt = min(32, M - i0);
        for (int k = 0; k < cnt; ++k) {
          const int cb = __shfl_sync(0xffffffffu, my_cb, k);
          const int t1 = __shfl_sync(0xffffffffu, my_t1, k);
          const int t2 = __shfl_sync(0xffffffffu, my_t2, k);
          if (lane == 0) {
            if (kc >= (uint32_t)S) mbar_wait(&empty[s], ph ^ 1);
            mbar_expect_tx(&full[s], bytes);
            bulk_load(bits_st(s), t1 >= 0 ? bits + (int64_t)t1 * 2 * TK : zero_bits, 2048, &full[s]);
            bulk_load(bits_st(s) + 2048, t2 >= 0 ? bits + (int64_t)t2 * 2 * TK : zero_bits, 2048, &full[s]);
            tma_load_4d(B_st(s), &tmB, &full[s], 0, n0, 0, cb);
          }
          ++kc;
          if (++s == S) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      const uint32_t idesc = idesc_i8(D * n_mma);
      const uint64_t bd0 = sdesc(smem_u32(B_st(0)), 16, 1024);
      const uint32_t st16 = (uint32_t)sh.stage_bytes >> 4;
      int s = 0, a = 0;
      uint32_t ph = 0, aph = 0;
      int it = 0;
      for (int t = blockIdx.x; t < total; t += gridDim.x, ++it) {
        const int item = t / sh.tiles_n;
        const int nst = pitem_pm[item + 1] - pitem_pm[item];
        if (it >= 1) mbar_wait(&tempty[0], (it - 1) & 1);   // single-buffered accumulators
        tc_fence_after();
        for (int st = 0; st < nst; ++st) {
          mbar_wait(&conv[a], aph);
          tc_fence_after();
          const uint32_t ta = tmem_base + kAcol + a * 64;
          const uint64_t bd = bd0 + (uint64_t)(s * st16);
          if (!(sh.dbg & 1)) {
#pragma unroll
            for (int j = 0; j < TK / 32; ++j) {
              const uint32_t acc = (st | j) ? 1u : 0u;
              tc_mma_i8_ts(tmem_base, ta + j * 8, bd + 2 * j, idesc, acc);
              tc_mma_i8_ts(tmem_base + (uint32_t)accw, ta + 32 + j * 8, bd + 2 * j, idesc, acc);
            }
          }
          tc_commit(&empty[s]);
          tc_commit(&aempty[a]);
          if (++s == S) { s = 0; ph ^= 1; }
          if (++a == SA) { a = 0; aph ^= 1; }
        }
        tc_commit(&tfull[0]);
      }
    }
  } else if (warp >= 4 && warp < 8) {
    const int r = threadIdx.x - 128;
    const uint32_t lane_off = (uint32_t)((warp & 3) * 32) << 16;
    int s = 0, a = 0;
    uint32_t ph = 0, aph = 0, kc = 0;
    for (int t = blockIdx.x; t < total; t += gridDim.x) {
      const int item = t / sh.tiles_n;
      const int nst = pitem_pm[item + 1] - pitem_pm[item];
      for (int st = 0; st < nst; ++st, ++kc) {
        mbar_wait(&full[s], ph);
        if (kc >= (uint32_t)SA) {
          mbar_wait(&aempty[a], aph ^ 1);
          tc_fence_after();
        }
#pragma unroll
        for (int tt = 0; tt < 2; ++tt) {
          const uint32_t bs = smem_u32(bits_st(s)) + tt * 2048 + r * 8;
          const uint2 h0 = lds64(bs), h1 = lds64(bs + 1024);
          const uint32_t w4[4] = {h0.x, h0.y, h1.x, h1.y};
          uint32_t v[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = (((w4[i >> 3] >> (4 * (i & 7))) & 15u) * 0x204081u) & 0x01010101u;
          tmem_st32u(tmem_base + lane_off + kAcol + a * 64 + tt * 32, v);
        }
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        tc_fence_before();
        mbar_arrive(&conv[a]);
        if (++s == S) { s = 0; ph ^= 1; }
        if (++a == SA) { a = 0; aph ^= 1; }
      }
    }
  } else if (warp >= 8) {
    const int q = warp & 3;
    int it = 0;
    for (int t = blockIdx.x; t < total; t += gridDim.x, ++it) {
      const int item = t / sh.tiles_n;
      const int64_t n0 = (int64_t)(t % sh.tiles_n) * n_mma;
      mbar_wait_sleep(&tfull[0], it & 1);
      tc_fence_after();
#pragma unroll 1
      for (int tt = 0; tt < 2; ++tt) {
        float* prow = part + ((int64_t)item * 2 * TK + tt * TK + q * 32 + lane) * sh.ldp + n0;
        for (int c0 = 0; c0 < n_mma; c0 += 32) {
          if (n0 + c0 >= sh.w) break;
          uint32_t dg[D][32];
          const uint32_t a0 = tmem_base + (uint32_t)(tt * accw) + ((uint32_t)(q * 32) << 16) + (uint32_t)c0;
#pragma unroll
          for (int d = 0; d < D; ++d) tmem_ld32(a0 + (uint32_t)(d * n_mma), dg[d]);
#pragma unroll
          for (int i = 0; i < 32; i += 4)
            if (n0 + c0 + i < sh.w) {
              const float4 cs = __ldg(reinterpret_cast<const float4*>(sh.colscale + n0 + c0 + i));
              float o[4];
#pragma unroll
              for (int u = 0; u < 4; ++u) {
                long long v = 0;
#pragma unroll
                for (int d = 0; d < D; ++d) v = v * 256 + (long long)(int)dg[d][i + u];
                o[u] = __ll2float_rn(v);
              }
              *reinterpret_cast<float4*>(prow + c0 + i) = make_float4(o[0] * cs.x, o[1] * cs.y, o[2] * cs.z, o[3] * cs.w);
            }
        }
      }
      tc_fence_before();
      mbar_arrive(&tempty[0]);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 2) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "n"(512));
  }
}

// int8 digit panels P_d[n][k] (row length K2 bytes; d = 0 the most
// significant) of y = s_k · X[hub_k][n] · 2^-e_n: D = 3 digits with the column
// maximum in [2^21, 2^22) (23-bit fixed point, fp32-class), D = 2 with it in
// [2^13, 2^14) (15-bit, the fast variant); colscale[n] = 2^e_n.
// Block: 128 k x 32 n, each thread 4 consecutive k.
template <int D>
__global__ void tile_panels_i8_kernel(const float* __restrict__ X, int64_t ldx, const int32_t* __restrict__ hub_ids,
                                      const float* __restrict__ scale, int64_t K2, int64_t w,
                                      const unsigned int* __restrict__ colmax, int8_t* __restrict__ pan,
                                      float* __restrict__ colscale) {
  __shared__ float t[128][33];
  __shared__ float inv[32];
  const int64_t k0 = (int64_t)blockIdx.x * 128, n0 = (int64_t)blockIdx.y * 32;
  if (threadIdx.y == 0) {
    const int64_t n = n0 + threadIdx.x;
    const float mx = n < w ? __uint_as_float(colmax[n]) : 0.f;
    const int e = mx > 0.f ? ilogbf(mx) - (8 * D - 3) : 0;
    inv[threadIdx.x] = ldexpf(1.f, -e);
    if (blockIdx.x == 0 && n < w) colscale[n] = ldexpf(1.f, e);
  }
  {
    const int64_t n = n0 + threadIdx.x;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      int32_t id[8];
      float sc[8], x[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int64_t k = k0 + threadIdx.y + 8 * u + 64 * h;
        id[u] = __ldg(hub_ids + k);
        sc[u] = __ldg(scale + k);
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) x[u] = (n < w) ? __ldg(X + (int64_t)id[u] * ldx + n) : 0.f;
#pragma unroll
      for (int u = 0; u < 8; ++u) t[threadIdx.y + 8 * u + 64 * h][threadIdx.x] = sc[u] * x[u];
    }
  }
  __syncthreads();
  for (int i = threadIdx.y; i < 32; i += 8) {
    const int64_t n = n0 + i;
    if (n >= w) break;
    const int kk = 4 * threadIdx.x;
    uint32_t q[D];
#pragma unroll
    for (int d = 0; d < D; ++d) q[d] = 0u;
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      int v = __float2int_rn(t[kk + u][i] * inv[i]);     // |v| <= 2^(8D-2)
      // balanced base-256 digits, least significant first: v = Σ d_j 256^j, d_j ∈ [-128, 127]
#pragma unroll
      for (int d = D - 1; d >= 0; --d) {
        const int dj = d == 0 ? v : ((v & 255) ^ 128) - 128;
        q[d] |= (uint32_t)(dj & 255) << (8 * u);
        v = (v - dj) >> 8;
      }
    }
    const int64_t o = n * K2 + k0 + kk;
#pragma unroll
    for (int d = 0; d < D; ++d) *reinterpret_cast<uint32_t*>(pan + (int64_t)d * w * K2 + o) = q[d];
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

// 4-D bf16 map over the three B panels P_p[n][k] (row length K2, panel p at
// p·w·K2): dims {64 (k within a 128-byte swizzle row), n, piece, k / 64}, box
// {64, n_mma, 3, HS}, so that one TMA lands [half][piece][n_mma][64] in smem
// with the 128-byte swizzle; rows n ≥ w read as zeros.
CUtensorMap panel_map(const void* base, int64_t K2, int64_t w, int n_mma, int HS, int np) {
  CUtensorMap m;
  cuuint64_t dims[4] = {(cuuint64_t)SK, (cuuint64_t)w, (cuuint64_t)np, (cuuint64_t)(K2 / SK)};
  cuuint64_t strides[3] = {(cuuint64_t)(K2 * 2), (cuuint64_t)(w * K2 * 2), (cuuint64_t)(SK * 2)};
  cuuint32_t box[4] = {(cuuint32_t)SK, (cuuint32_t)n_mma, (cuuint32_t)np, (cuuint32_t)HS};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = encode()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(base), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(RDM_ERR_CUDA, "cuTensorMapEncodeTiled (panels) failed (" + std::to_string((int)r) + ")");
  return m;
}

// 4-D int8 map over the three digit panels P_d[n][k] (row length K2 bytes,
// panel d at d·w·K2): dims {128 (k within a tile = one 128-byte swizzle row),
// n, digit, k / 128}, box {128, n_mma, 3, 1}: one TMA lands [digit][n_mma][128].
CUtensorMap panel_map_i8(const void* base, int64_t K2, int64_t w, int n_mma, int D) {
  CUtensorMap m;
  cuuint64_t dims[4] = {(cuuint64_t)TK, (cuuint64_t)w, (cuuint64_t)D, (cuuint64_t)(K2 / TK)};
  cuuint64_t strides[3] = {(cuuint64_t)K2, (cuuint64_t)(w * K2), (cuuint64_t)TK};
  cuuint32_t box[4] = {(cuuint32_t)TK, (cuuint32_t)n_mma, (cuuint32_t)D, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = encode()(&m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, const_cast<void*>(base), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(RDM_ERR_CUDA, "cuTensorMapEncodeTiled (int8 panels) failed (" + std::to_string((int)r) + ")");
  return m;
}

CUtensorMap stacked_map(const void* base, int64_t K2, int64_t rows, int n_mma) {
  CUtensorMap m;
  cuuint64_t dims[2] = {(cuuint64_t)K2, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)(K2 * 2)};
  cuuint32_t box[2] = {(cuuint32_t)SK, (cuuint32_t)n_mma};
  cuuint32_t es[2] = {1, 1};
  CUresult r = encode()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) throw Error(RDM_ERR_CUDA, "cuTensorMapEncodeTiled (stacked) failed (" + std::to_string((int)r) + ")");
  return m;
}

// Per-call cost model (B200, calibrated on the Reddit-shaped graph,
// profiles/r1_hub_tiles_reddit.txt): a CSR entry costs ≈ 24 ps·(w/128)^0.55
// (L2-gather bound), a tile ≈ ceil(w/128)·(4.5 + 5.2·min(w,128)/128) ns (bit
// expansion + 3 bf16 MMA pieces per 128-wide chunk), plus ≈ 20 µs per call.
double csr_entry_s(int64_t w) { return 24e-12 * std::pow((double)w / 128.0, 0.55); }
double tile_s(int64_t w, int np = 3) {
  if (np == kPiecesI8 || np == kPiecesI8x2)   // int8 digits, 64-wide passes (Reddit-shaped: ≈ 3 ns / pass)
    return (double)ceil_div(w, I8_NMAX) * (1.2e-9 + (np == kPiecesI8 ? 2.0e-9 : 1.4e-9) *
                                                      (double)std::min<int64_t>(w, I8_NMAX) / I8_NMAX);
  return (double)ceil_div(w, 128) * (4.5e-9 + 5.2e-9 * np / 3.0 * (double)std::min<int64_t>(w, 128) / 128.0);
}
}  // namespace

// The int8 tiles run in row-block pairs with RDM_TILE_PAIRS=1 (off by
// default: measured no faster — Reddit-shaped w = 128 1.235 vs 1.232 ms per
// call, w = 16 0.417 vs 0.387, products-shaped w = 256 8.30 vs 8.41 ms; the
// single kernel is bound by the tensor pipe's int8 rate at N = 3·64, not by
// the panel ingress the pairs halve, profiles/r2_tile_pairs.txt).
bool tiles_paired() {
  const char* e = getenv("RDM_TILE_PAIRS");
  return e && atoi(e);
}

bool hub_tiles_pay(const Core& c, int64_t w, int np) {
  if (!c.n_tiles) return false;
  if (c.forced) return true;
  return (double)c.nnz * csr_entry_s(w) > (double)c.n_tiles * tile_s(w, np) + 20e-6;
}

// int8 digits (np == kPiecesI8: 3, kPiecesI8x2: 2): column maxima, digit
// panels, hub_tile_i8_kernel<D>.
// tiles per stage of hub_tile_i8_kernel (RDM_TILE_TPS=1 / 2 for experiments)
int tile_tps() {
  const char* e = getenv("RDM_TILE_TPS");
  return e && atoi(e) == 1 ? 1 : 2;
}

void hub_tiles_product_i8(rdm_ctx* ctx, const Core& c, const float* X, int64_t ldx, int64_t w, float* part,
                          int64_t ldp, int D) {
  const int64_t K2 = c.K2;
  int8_t* pan = reinterpret_cast<int8_t*>(ensure_ws(ctx->ws_core_b, (size_t)D * w * K2));
  const int64_t w4 = (w + 3) / 4 * 4;
  float* cs = ensure_ws(ctx->ws_tile_cs, (size_t)2 * w4 * sizeof(float));
  unsigned int* cmax = reinterpret_cast<unsigned int*>(cs + w4);
  RDM_CUDA(cudaMemsetAsync(cmax, 0, w * sizeof(unsigned int), ctx->stream));
  RDM_CUDA(cudaMemsetAsync(cs, 0, w4 * sizeof(float), ctx->stream));
  dim3 mg((unsigned)ceil_div(K2, 256), (unsigned)ceil_div(w, 32));
  tile_colmax_kernel<<<mg, dim3(32, 8), 0, ctx->stream>>>(X, ldx, c.hub_ids->as<int32_t>(), c.scale->as<float>(),
                                                         K2, w, cmax);
  RDM_LAUNCHED(ctx);
  dim3 pg((unsigned)(K2 / TK), (unsigned)ceil_div(w, 32));
  auto pk = D == 3 ? tile_panels_i8_kernel<3> : tile_panels_i8_kernel<2>;
  pk<<<pg, dim3(32, 8), 0, ctx->stream>>>(X, ldx, c.hub_ids->as<int32_t>(), c.scale->as<float>(), K2, w, cmax, pan,
                                          cs);
  RDM_LAUNCHED(ctx);
  TileShape sh{};
  sh.n_mma = (int)std::min<int64_t>(I8_NMAX, ((w + 15) / 16) * 16);
  sh.tiles_n = (int)ceil_div(w, sh.n_mma);
  sh.n_items = (int)c.n_items;
  sh.w = w;
  sh.ldp = ldp;
  sh.R = 1;
  sh.HS = 1;
  sh.acc_cols = (D * sh.n_mma + 31) / 32 * 32;
  const int TP = tile_tps();   // (3 per stage at w = 41: no change, 0.630 ms per call)
  sh.stage_bytes = (TP * (D * sh.n_mma * 128 + 2048) + 1023) / 1024 * 1024;
  const int avail = kSmemBudget - 1024 - 1024;
  sh.S = std::min(32, avail / sh.stage_bytes);
  sh.SA = std::min(8, (512 - 2 * sh.acc_cols) / (32 * TP));
  sh.dbg = getenv("RDM_TILE_DBG") ? atoi(getenv("RDM_TILE_DBG")) : 0;
  sh.colscale = cs;
  RDM_CHECK_ARG(sh.S >= 2 && sh.SA >= 2, "hub tiles (int8): TMEM/smem budget");
  const CUtensorMap tb = panel_map_i8(pan, K2, w, (sh.dbg & 8) ? sh.n_mma / 2 : sh.n_mma, D);
  if (tiles_paired()) {
    // two row blocks per panel load (hub_tile_i8_pair_kernel)
    TileShape ps = sh;
    ps.n_items = (int)c.n_pitems;
    ps.acc_cols = (2 * D * sh.n_mma + 31) / 32 * 32;
    ps.stage_bytes = (D * sh.n_mma * 128 + 4096 + 1023) / 1024 * 1024;
    ps.S = std::min(32, (kSmemBudget - 1024 - 1024) / ps.stage_bytes);
    ps.SA = std::min(8, (512 - ps.acc_cols) / 64);
    RDM_CHECK_ARG(ps.S >= 2 && ps.SA >= 2, "hub tiles (int8 pairs): TMEM/smem budget");
    const int psmem = ps.S * ps.stage_bytes + 1024 + 1024;
    const int64_t ptotal = c.n_pitems * ps.tiles_n;
    const unsigned pgrid = (unsigned)std::min<int64_t>(ptotal, ctx->num_sms);
    auto pk = D == 3 ? hub_tile_i8_pair_kernel<3> : hub_tile_i8_pair_kernel<2>;
    RDM_CUDA(cudaFuncSetAttribute(pk, cudaFuncAttributeMaxDynamicSharedMemorySize, psmem));
    pk<<<pgrid, 384, psmem, ctx->stream>>>(tb, c.tiles->as<uint64_t>(), c.zero_bits->as<uint64_t>(),
                                           c.pm_cb->as<int32_t>(), c.pm_t1->as<int32_t>(),
                                           c.pm_t2->as<int32_t>(), c.pitem_pm->as<int32_t>(), part, ps);
    RDM_LAUNCHED(ctx);
    return;
  }
  const int smem = sh.S * sh.stage_bytes + 1024 + 1024;
  const int64_t total = c.n_items * sh.tiles_n;
  const unsigned grid = (unsigned)std::min<int64_t>(total, ctx->num_sms);
  auto kern = D == 3 ? (TP == 2 ? hub_tile_i8_kernel<3, 2> : hub_tile_i8_kernel<3, 1>)
                     : (TP == 2 ? hub_tile_i8_kernel<2, 2> : hub_tile_i8_kernel<2, 1>);
  RDM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  kern<<<grid, 384, smem, ctx->stream>>>(tb, c.tiles->as<uint64_t>(), c.zero_bits->as<uint64_t>(),
                                         c.tile_cb->as<int32_t>(), c.item_tb->as<int32_t>(), part, sh);
  RDM_LAUNCHED(ctx);
}

void hub_tiles_product(rdm_ctx* ctx, const Core& c, const float* X, int64_t ldx, int64_t w, float* part,
                       int64_t ldp, int np) {
  if (np == kPiecesI8) return hub_tiles_product_i8(ctx, c, X, ldx, w, part, ldp, 3);
  if (np == kPiecesI8x2) return hub_tiles_product_i8(ctx, c, X, ldx, w, part, ldp, 2);
  RDM_CHECK_ARG(np >= 1 && np <= 3, "hub tiles: 1, 2 or 3 pieces");
  const int64_t K2 = c.K2;
  __nv_bfloat16* pan = reinterpret_cast<__nv_bfloat16*>(ensure_ws(ctx->ws_core_b, (size_t)np * w * K2 * 2));
  dim3 pg((unsigned)(K2 / 64), (unsigned)ceil_div(w, 32));
  float* colscale = nullptr;
  if (np == 2) {
    // column scales: max |s·X| per column, then fp16 hi / lo pieces
    const int64_t w4 = (w + 3) / 4 * 4;
    float* cs = ensure_ws(ctx->ws_tile_cs, (size_t)2 * w4 * sizeof(float));
    unsigned int* cmax = reinterpret_cast<unsigned int*>(cs + w4);
    RDM_CUDA(cudaMemsetAsync(cmax, 0, w * sizeof(unsigned int), ctx->stream));
    RDM_CUDA(cudaMemsetAsync(cs, 0, w4 * sizeof(float), ctx->stream));
    dim3 mg((unsigned)ceil_div(K2, 256), (unsigned)ceil_div(w, 32));
    tile_colmax_kernel<<<mg, dim3(32, 8), 0, ctx->stream>>>(X, ldx, c.hub_ids->as<int32_t>(), c.scale->as<float>(),
                                                           K2, w, cmax);
    RDM_LAUNCHED(ctx);
    tile_panels_f16_kernel<<<pg, dim3(32, 8), 0, ctx->stream>>>(
        X, ldx, c.hub_ids->as<int32_t>(), c.scale->as<float>(), K2, w, cmax, reinterpret_cast<__half*>(pan),
        reinterpret_cast<__half*>(pan + w * K2), cs);
    RDM_LAUNCHED(ctx);
    colscale = cs;
  } else {
    tile_panels_kernel<<<pg, dim3(32, 8), 0, ctx->stream>>>(X, ldx, c.hub_ids->as<int32_t>(), c.scale->as<float>(),
                                                          K2, w, pan, pan + w * K2, pan + 2 * w * K2, np);
    RDM_LAUNCHED(ctx);
  }
  TileShape sh;
  sh.n_mma = (int)std::min<int64_t>(128, ((w + 15) / 16) * 16);
  sh.tiles_n = (int)ceil_div(w, 128);
  sh.n_items = (int)c.n_items;
  sh.w = w;
  sh.ldp = ldp;
  sh.R = sh.n_mma <= 64 ? (sh.n_mma <= 16 ? 2 : 1) : 0;
  if (const char* e = getenv("RDM_TILE_R")) sh.R = sh.n_mma <= 64 ? std::max(0, std::min(4, atoi(e))) : 0;
  sh.acc_cols = (int)((sh.R ? sh.R * np * sh.n_mma : sh.n_mma) + 31) / 32 * 32;
  // whole tiles per stage when the stage stays small (narrow slices: halves
  // the per-stage fixed cost), else 64-wide k halves
  sh.HS = np * sh.n_mma * 256 + 2048 <= 50 * 1024 ? 2 : 1;
  if (const char* e = getenv("RDM_TILE_HS")) sh.HS = atoi(e) == 2 ? 2 : 1;
  sh.stage_bytes = sh.HS * (np * sh.n_mma * 128 + 1024);
  const int avail = kSmemBudget - 1024 - 1024 - 4096;   // align, barriers, LUT
  sh.S = std::min(32, avail / sh.stage_bytes);
  sh.SA = std::min(8, (512 - 2 * sh.acc_cols) / (32 * sh.HS));
  sh.dbg = getenv("RDM_TILE_DBG") ? atoi(getenv("RDM_TILE_DBG")) : 0;
  sh.colscale = colscale;
  RDM_CHECK_ARG(sh.S >= 2 && sh.SA >= 2, "hub tiles: TMEM/smem budget");
  const CUtensorMap tb = panel_map(pan, K2, w, sh.n_mma, sh.HS, np);
  // the three panels stacked as one 3w x K2 matrix: rows past a panel's w
  // only feed accumulator columns ≥ w, which are never stored
  const CUtensorMap tb2 = stacked_map(pan, K2, np * w, sh.n_mma);
  const int smem = sh.S * sh.stage_bytes + 1024 + 1024 + 4096;
  const int64_t total = c.n_items * sh.tiles_n;
  const unsigned grid = (unsigned)std::min<int64_t>(total, ctx->num_sms);
  auto kern = np == 3 ? (sh.HS == 2 ? hub_tile_kernel<2, 3> : hub_tile_kernel<1, 3>)
             : np == 2 ? (sh.HS == 2 ? hub_tile_kernel<2, 2> : hub_tile_kernel<1, 2>)
                       : (sh.HS == 2 ? hub_tile_kernel<2, 1> : hub_tile_kernel<1, 1>);
  RDM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  kern<<<grid, 384, smem, ctx->stream>>>(tb, tb2, c.tiles->as<uint64_t>(), c.tile_cb->as<int32_t>(),
                                         c.item_tb->as<int32_t>(), part, sh);
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
  // factorisation â_ij = r_i · c_j on every moved entry (any rank-1 scaling of
  // a 0/1 block: the symmetric GCN normalisation s_i s_j, the row-normalised
  // D^-1 (A+I) (r = 1/deg, c = 1), unit values, …).  r and c are found by a
  // walk over the moved entries (a row fixes the columns it reaches, a column
  // fixes the rows that reach it; the pattern is symmetric), every component
  // anchored at r = 1, then every moved entry is checked to 2^-21 relative.
  std::vector<double> rs(K2, 0.0), cs(K2, 0.0);   // by rank
  auto in_tile = [&](int64_t ri, int64_t rj) {
    return rj < K2 && tile_id[(size_t)(ri / TK) * nrb + rj / TK] >= 0;
  };
  auto verify = [&]() {
    for (int64_t i = 0; i < n; ++i) {
      const int64_t ri = rank[i];
      if (ri >= K2) continue;
      for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
        const int64_t rj = rank[col[j]];
        if (!in_tile(ri, rj)) continue;
        const double f = rs[ri] * cs[rj];
        if (f == 0.0 || !(std::fabs((double)val[j] - f) <= std::ldexp(std::fabs(f), -21))) return false;
      }
    }
    return true;
  };
  // closed forms first (exact factors): s s (GCN), 1/deg · 1 (row-normalised),
  // 1 · 1/deg (column-normalised), 1 · 1
  bool ok = false;
  for (int hyp = 0; hyp < 4 && !ok; ++hyp) {
    for (int64_t k = 0; k < K2; ++k) {
      const double d = (double)(rp[order[k] + 1] - rp[order[k]]);
      const double s = 1.0 / std::sqrt(d);
      rs[k] = hyp == 0 ? s : hyp == 1 ? 1.0 / d : 1.0;
      cs[k] = hyp == 0 ? s : hyp == 2 ? 1.0 / d : 1.0;
    }
    ok = verify();
  }
  if (!ok) {
    // any other rank-1 scaling: a walk over the moved entries (a row fixes the
    // columns it reaches, a column fixes the rows that reach it; the pattern is
    // symmetric), each component anchored at r = 1, then two refinement sweeps
    // (geometric means of the ratios: the walk's rounding errors grow with the
    // path length) before the check
    auto value = [&](int64_t i, int64_t j) -> double {   // a_ij (vertex ids), found in row i
      const int32_t* b = col + rp[i];
      const int32_t* e = col + rp[i + 1];
      const int32_t* f = std::lower_bound(b, e, (int32_t)j);
      return (f != e && *f == (int32_t)j) ? (double)val[f - col] : std::nan("");
    };
    std::fill(rs.begin(), rs.end(), 0.0);
    std::fill(cs.begin(), cs.end(), 0.0);
    std::vector<char> rset(K2, 0), cset(K2, 0);
    std::vector<int64_t> queue;   // >= 0: row rank, < 0: -(column rank) - 1
    ok = true;
    for (int64_t root = 0; root < K2 && ok; ++root) {
      if (rset[root]) continue;
      rs[root] = 1.0;
      rset[root] = 1;
      queue.assign(1, root);
      while (!queue.empty() && ok) {
        const int64_t q = queue.back();
        queue.pop_back();
        if (q >= 0) {
          const int64_t i = order[q];
          for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
            const int64_t rj = rank[col[j]];
            if (!in_tile(q, rj) || cset[rj]) continue;
            cs[rj] = (double)val[j] / rs[q];
            cset[rj] = 1;
            queue.push_back(-rj - 1);
          }
        } else {
          const int64_t cj = -q - 1, v = order[cj];
          for (int64_t k = rp[v]; k < rp[v + 1]; ++k) {
            const int64_t rk = rank[col[k]];
            if (rk >= K2 || rset[rk] || !in_tile(rk, cj)) continue;
            const double a = value(col[k], v);
            if (!(a == a) || a == 0.0 || cs[cj] == 0.0) { ok = false; break; }
            rs[rk] = a / cs[cj];
            rset[rk] = 1;
            queue.push_back(rk);
          }
        }
      }
    }
    for (int sweep = 0; sweep < 2 && ok; ++sweep) {
      std::vector<double> lr(K2, 0.0), lc(K2, 0.0);
      std::vector<int64_t> nr(K2, 0), nc(K2, 0);
      for (int64_t i = 0; i < n; ++i) {   // rows from the columns
        const int64_t ri = rank[i];
        if (ri >= K2) continue;
        for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
          const int64_t rj = rank[col[j]];
          if (!in_tile(ri, rj) || val[j] <= 0.f || cs[rj] <= 0.0) continue;
          lr[ri] += std::log((double)val[j] / cs[rj]);
          nr[ri]++;
        }
      }
      for (int64_t k = 0; k < K2; ++k)
        if (nr[k]) rs[k] = std::exp(lr[k] / nr[k]);
      for (int64_t i = 0; i < n; ++i) {   // columns from the rows
        const int64_t ri = rank[i];
        if (ri >= K2) continue;
        for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
          const int64_t rj = rank[col[j]];
          if (!in_tile(ri, rj) || val[j] <= 0.f || rs[ri] <= 0.0) continue;
          lc[rj] += std::log((double)val[j] / rs[ri]);
          nc[rj]++;
        }
      }
      for (int64_t k = 0; k < K2; ++k)
        if (nc[k]) cs[k] = std::exp(lc[k] / nc[k]);
    }
    ok = ok && verify();
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
  // tiles as bits (bits[tile][half][row] = u64, bit kk = column half·64 + kk),
  // filled one row block at a time; an entry whose cell is already set (a
  // duplicate (i, j) in the CSR) stays in the residual CSR.
  c.tiles.reset(new DevBuf((size_t)n_tiles * TK * TK / 8));
  std::vector<uint8_t> tin(nnz, 0);
  std::vector<uint64_t> buf;
  for (int64_t rb = 0; rb < c.n_rb; ++rb) {
    const int64_t t0 = rb_first[rb], T = rb_first[rb + 1] - t0;
    if (!T) continue;
    buf.assign((size_t)T * 2 * TK, 0);
    for (int64_t r = 0; r < TK; ++r) {
      const int64_t v = order[rb * TK + r];
      for (int64_t j = rp[v]; j < rp[v + 1]; ++j) {
        const int64_t rj = rank[col[j]];
        if (rj >= K2) continue;
        const int64_t id = tile_id[(size_t)rb * nrb + rj / TK];
        if (id < 0) continue;
        const int64_t cc = rj % TK;
        uint64_t& word = buf[(size_t)(id - t0) * 2 * TK + (cc / SK) * TK + r];
        const uint64_t bit = 1ull << (cc % SK);
        if (word & bit) continue;
        word |= bit;
        tin[j] = 1;
      }
    }
    RDM_CUDA(cudaMemcpy(c.tiles->as<uint64_t>() + (size_t)t0 * 2 * TK, buf.data(), buf.size() * 8,
                        cudaMemcpyHostToDevice));
  }
  std::vector<int64_t> rrp(n + 1, 0);
  for (int64_t i = 0; i < n; ++i) {
    int64_t keep = 0;
    for (int64_t j = rp[i]; j < rp[i + 1]; ++j) keep += !tin[j];
    rrp[i + 1] = rrp[i] + keep;
  }
  const int64_t rnnz = rrp[n];
  c.nnz = nnz - rnnz;
  std::vector<int32_t> rcol(std::max<int64_t>(rnnz, 1));
  std::vector<float> rval(std::max<int64_t>(rnnz, 1));
  for (int64_t i = 0; i < n; ++i) {
    int64_t o = rrp[i];
    for (int64_t j = rp[i]; j < rp[i + 1]; ++j)
      if (!tin[j]) {
        rcol[o] = col[j];
        rval[o] = val[j];
        ++o;
      }
  }
  // pair items (int8 kernel): row blocks 2p and 2p+1 against ONE panel load
  // per column block in the union of their tiles (merged in column order; a
  // row block without a tile there multiplies a zero tile); runs of at most
  // `chunk` merged entries, ≈ 4 items per SM
  std::vector<int32_t> pm_cb, pm_t1, pm_t2, pitem_pm, pair_item;
  {
    const int64_t n_pairs = (c.n_rb + 1) / 2;
    std::vector<int64_t> pm_first(n_pairs + 1, 0);
    for (int64_t p = 0; p < n_pairs; ++p) {
      pm_first[p] = (int64_t)pm_cb.size();
      const int64_t r1 = 2 * p, r2 = 2 * p + 1;
      int64_t i = rb_first[r1], ie = rb_first[r1 + 1];
      int64_t j = r2 < c.n_rb ? rb_first[r2] : 0, je = r2 < c.n_rb ? rb_first[r2 + 1] : 0;
      while (i < ie || j < je) {
        const int32_t ci = i < ie ? tile_cb[i] : INT32_MAX, cj = j < je ? tile_cb[j] : INT32_MAX;
        const int32_t cb = std::min(ci, cj);
        pm_cb.push_back(cb);
        pm_t1.push_back(ci == cb ? (int32_t)i++ : -1);
        pm_t2.push_back(cj == cb ? (int32_t)j++ : -1);
      }
    }
    pm_first[n_pairs] = (int64_t)pm_cb.size();
    const int64_t pchunk = std::max<int64_t>(4, ceil_div((int64_t)pm_cb.size(), (int64_t)ctx->num_sms * 4));
    pair_item.assign(n_pairs + 1, 0);
    for (int64_t p = 0; p < n_pairs; ++p) {
      pair_item[p] = (int32_t)pitem_pm.size();
      const int64_t m0 = pm_first[p], M = pm_first[p + 1] - m0;
      const int64_t nit = ceil_div(M, pchunk);
      for (int64_t k = 0; k < nit; ++k) pitem_pm.push_back((int32_t)(m0 + M * k / nit));
    }
    pair_item[n_pairs] = (int32_t)pitem_pm.size();
    c.n_pairs = n_pairs;
    c.n_pitems = (int64_t)pitem_pm.size();
    pitem_pm.push_back((int32_t)pm_cb.size());
  }
  std::vector<float> sc(c.K2), sr(c.K2);
  for (int64_t k = 0; k < c.K2; ++k) {
    sc[k] = (float)cs[k];   // column scale of hub slot k (panels)
    sr[k] = (float)rs[k];   // row scale (the SpMM epilogue)
  }
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
  up(c.rscale, sr.data(), sr.size() * 4);
  up(c.pm_cb, pm_cb.data(), pm_cb.size() * 4);
  up(c.pm_t1, pm_t1.data(), pm_t1.size() * 4);
  up(c.pm_t2, pm_t2.data(), pm_t2.size() * 4);
  up(c.pitem_pm, pitem_pm.data(), pitem_pm.size() * 4);
  up(c.pair_item, pair_item.data(), pair_item.size() * 4);
  {
    std::vector<uint64_t> z(2 * TK, 0);
    up(c.zero_bits, z.data(), z.size() * 8);
  }
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
