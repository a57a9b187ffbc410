// redist.cu — divide / merge kernels of the row↔column redistribution.
//
// PAPER.md Fig. 7 / L212: "each processor then divides the data it owns into
// P vertical chunks (the divide step) ... each processor merges its chunks
// (Merge step)".  With the library's layouts (rdm.h) a column slice of rank q
// is N x ld_q row-major, so the block rank p owes rank q in a row→col
// redistribution (its rows × q's columns) is a contiguous r_p x ld_q array
// that lands verbatim at rows [lo_p, hi_p) of q's column slice: only the
// SENDER permutes (pack = divide), the receiver's merge is free.  In col→row
// the sender's blocks are contiguous row ranges of its column slice (free) and
// the RECEIVER permutes (unpack = merge).  The self block never leaves the
// GPU: pack writes it straight into the destination slice, unpack reads it
// straight from the source slice.
//
// A source row of ld_row = roundup4(f) floats is exactly the concatenation of
// the P blocks' rows (ld_q floats each, granule-aligned partition), so both
// kernels are a streaming float4 copy with a per-element block lookup.
#include <cuda_bf16.h>

#include "internal.h"

namespace rdm {
namespace {

struct Tab {
  int P;
  int64_t c4_lo[BlockTable::kMax + 1];  // first float4 column of block q in the row
  const float* src[BlockTable::kMax];
  float* dst[BlockTable::kMax];
};

__device__ __forceinline__ int find_block(const Tab& t, int64_t c4) {
  int q = 0;
  while (q + 1 < t.P && t.c4_lo[q + 1] <= c4) ++q;
  return q;
}

// row slice (rows x ld_row) → blocks (rows x ld_q each)
__global__ void pack_kernel(const float* __restrict__ row_slice, int64_t ld_row4, int64_t rows,
                            Tab t) {
  const int64_t total = rows * ld_row4;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total;
       g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = g / ld_row4, c4 = g % ld_row4;
    const int q = find_block(t, c4);
    const int64_t ld_q4 = t.c4_lo[q + 1] - t.c4_lo[q];
    const float4 v = __ldcs(reinterpret_cast<const float4*>(row_slice) + g);
    reinterpret_cast<float4*>(t.dst[q])[i * ld_q4 + (c4 - t.c4_lo[q])] = v;
  }
}

// blocks (rows x ld_q each) → row slice (rows x ld_row)
__global__ void unpack_kernel(float* __restrict__ row_slice, int64_t ld_row4, int64_t rows, Tab t) {
  const int64_t total = rows * ld_row4;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total;
       g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = g / ld_row4, c4 = g % ld_row4;
    const int q = find_block(t, c4);
    const int64_t ld_q4 = t.c4_lo[q + 1] - t.c4_lo[q];
    const float4 v = __ldcs(reinterpret_cast<const float4*>(t.src[q]) + i * ld_q4 + (c4 - t.c4_lo[q]));
    reinterpret_cast<float4*>(row_slice)[g] = v;
  }
}

Tab make_tab(int P, const BlockTable& bt) {
  Tab t{};
  t.P = P;
  int64_t acc = 0;
  for (int q = 0; q < P; ++q) {
    t.c4_lo[q] = acc;
    acc += bt.ld[q] / 4;
    t.src[q] = bt.src[q];
    t.dst[q] = bt.dst[q];
  }
  t.c4_lo[P] = acc;
  return t;
}

unsigned grid_for(rdm_ctx* ctx, int64_t total) {
  const int64_t want = ceil_div(total, 256);
  return (unsigned)std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)ctx->num_sms * 16));
}

}  // namespace

void pack_rows(rdm_ctx* ctx, const float* row_slice, int64_t ld_row, int64_t rows, int P,
               const BlockTable& bt) {
  if (rows == 0 || ld_row == 0) return;
  Tab t = make_tab(P, bt);
  RDM_CHECK_ARG(t.c4_lo[P] * 4 == ld_row, "pack: block widths do not tile the row");
  const int64_t total = rows * (ld_row / 4);
  pack_kernel<<<grid_for(ctx, total), 256, 0, ctx->stream>>>(row_slice, ld_row / 4, rows, t);
  RDM_LAUNCHED(ctx);
}

void unpack_rows(rdm_ctx* ctx, float* row_slice, int64_t ld_row, int64_t rows, int P,
                 const BlockTable& bt) {
  if (rows == 0 || ld_row == 0) return;
  Tab t = make_tab(P, bt);
  RDM_CHECK_ARG(t.c4_lo[P] * 4 == ld_row, "unpack: block widths do not tile the row");
  const int64_t total = rows * (ld_row / 4);
  unpack_kernel<<<grid_for(ctx, total), 256, 0, ctx->stream>>>(row_slice, ld_row / 4, rows, t);
  RDM_LAUNCHED(ctx);
}

// ------------------------------------------------------------ bf16 wire
// RDM_PREC_FAST inside the executor: the redistribution carries bf16 (half the
// (P−1)/P·N·f·4 bytes of L142), rounded once (RNE) at the sender; every rank's
// blocks, its own included, hold bf16-exact values afterwards, so the result
// does not depend on the partition.  A 128-bit bf16 vector is 8 columns;
// ld values are multiples of 4, so blocks are handled in 4-column units
// (uint2 = 4 bf16).
namespace {
__device__ __forceinline__ uint2 to_bf4(float4 v) {
  __nv_bfloat162 a = __floats2bfloat162_rn(v.x, v.y), b = __floats2bfloat162_rn(v.z, v.w);
  return make_uint2(*reinterpret_cast<uint32_t*>(&a), *reinterpret_cast<uint32_t*>(&b));
}
__device__ __forceinline__ float4 from_bf4(uint2 u) {
  return make_float4(__uint_as_float(u.x << 16), __uint_as_float(u.x & 0xFFFF0000u), __uint_as_float(u.y << 16),
                     __uint_as_float(u.y & 0xFFFF0000u));
}

struct TabH {
  int P, self;
  int64_t c4_lo[BlockTable::kMax + 1];
  uint2* dst[BlockTable::kMax];   // bf16 blocks (rows x ld_q), null for the self block
  float* self_dst;                // self block: fp32, straight into the column slice (ld_self)
  const uint2* src[BlockTable::kMax];
  const float* self_src;
  int64_t ld_self4;
};

__device__ __forceinline__ int find_block_h(const TabH& t, int64_t c4) {
  int q = 0;
  while (q + 1 < t.P && t.c4_lo[q + 1] <= c4) ++q;
  return q;
}

// row slice (fp32) → bf16 blocks; the self block → fp32(bf16(x)) in place
__global__ void pack_bf16_kernel(const float* __restrict__ row_slice, int64_t ld_row4, int64_t rows, TabH t) {
  const int64_t total = rows * ld_row4;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total; g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = g / ld_row4, c4 = g % ld_row4;
    const int q = find_block_h(t, c4);
    const int64_t ld_q4 = t.c4_lo[q + 1] - t.c4_lo[q];
    const uint2 h = to_bf4(__ldcs(reinterpret_cast<const float4*>(row_slice) + g));
    if (q == t.self)
      reinterpret_cast<float4*>(t.self_dst)[i * t.ld_self4 + (c4 - t.c4_lo[q])] = from_bf4(h);
    else
      t.dst[q][i * ld_q4 + (c4 - t.c4_lo[q])] = h;
  }
}

// bf16 blocks + fp32 self block → row slice (fp32)
__global__ void unpack_bf16_kernel(float* __restrict__ row_slice, int64_t ld_row4, int64_t rows, TabH t) {
  const int64_t total = rows * ld_row4;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total; g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = g / ld_row4, c4 = g % ld_row4;
    const int q = find_block_h(t, c4);
    const int64_t ld_q4 = t.c4_lo[q + 1] - t.c4_lo[q];
    float4 v;
    if (q == t.self)
      v = from_bf4(to_bf4(__ldcs(reinterpret_cast<const float4*>(t.self_src) + i * t.ld_self4 + (c4 - t.c4_lo[q]))));
    else
      v = from_bf4(__ldcs(t.src[q] + i * ld_q4 + (c4 - t.c4_lo[q])));
    reinterpret_cast<float4*>(row_slice)[g] = v;
  }
}

// column slice rows [0, n) except [skip_lo, skip_hi): fp32 ↔ bf16 staging of
// the same shape (n x ld, 4-column units)
__global__ void narrow_cols_kernel(const float* __restrict__ col, int64_t n4, int64_t skip_lo4, int64_t skip_hi4,
                                   uint2* __restrict__ stage) {
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < n4; g += (int64_t)gridDim.x * blockDim.x)
    if (g < skip_lo4 || g >= skip_hi4) stage[g] = to_bf4(__ldcs(reinterpret_cast<const float4*>(col) + g));
}
__global__ void widen_cols_kernel(const uint2* __restrict__ stage, int64_t n4, int64_t skip_lo4, int64_t skip_hi4,
                                  float* __restrict__ col) {
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < n4; g += (int64_t)gridDim.x * blockDim.x)
    if (g < skip_lo4 || g >= skip_hi4) reinterpret_cast<float4*>(col)[g] = from_bf4(__ldcs(stage + g));
}

TabH make_tabh(int P, int self, const BlockTable& bt) {
  TabH t{};
  t.P = P;
  t.self = self;
  int64_t acc = 0;
  for (int q = 0; q < P; ++q) {
    t.c4_lo[q] = acc;
    acc += bt.ld[q] / 4;
  }
  t.c4_lo[P] = acc;
  return t;
}
}  // namespace

void pack_rows_bf16(rdm_ctx* ctx, const float* row_slice, int64_t ld_row, int64_t rows, int P, int self,
                    const BlockTable& bt, float* self_dst, int64_t ld_self) {
  if (rows == 0 || ld_row == 0) return;
  TabH t = make_tabh(P, self, bt);
  RDM_CHECK_ARG(t.c4_lo[P] * 4 == ld_row, "pack (bf16): block widths do not tile the row");
  for (int q = 0; q < P; ++q) t.dst[q] = reinterpret_cast<uint2*>(bt.dst[q]);
  t.self_dst = self_dst;
  t.ld_self4 = ld_self / 4;
  const int64_t total = rows * (ld_row / 4);
  pack_bf16_kernel<<<grid_for(ctx, total), 256, 0, ctx->stream>>>(row_slice, ld_row / 4, rows, t);
  RDM_LAUNCHED(ctx);
}

void unpack_rows_bf16(rdm_ctx* ctx, float* row_slice, int64_t ld_row, int64_t rows, int P, int self,
                      const BlockTable& bt, const float* self_src, int64_t ld_self) {
  if (rows == 0 || ld_row == 0) return;
  TabH t = make_tabh(P, self, bt);
  RDM_CHECK_ARG(t.c4_lo[P] * 4 == ld_row, "unpack (bf16): block widths do not tile the row");
  for (int q = 0; q < P; ++q) t.src[q] = reinterpret_cast<const uint2*>(bt.src[q]);
  t.self_src = self_src;
  t.ld_self4 = ld_self / 4;
  const int64_t total = rows * (ld_row / 4);
  unpack_bf16_kernel<<<grid_for(ctx, total), 256, 0, ctx->stream>>>(row_slice, ld_row / 4, rows, t);
  RDM_LAUNCHED(ctx);
}

void narrow_cols(rdm_ctx* ctx, const float* col, int64_t n, int64_t ld, int64_t skip_lo, int64_t skip_hi,
                 void* stage) {
  const int64_t n4 = n * ld / 4;
  if (!n4) return;
  narrow_cols_kernel<<<grid_for(ctx, n4), 256, 0, ctx->stream>>>(col, n4, skip_lo * ld / 4, skip_hi * ld / 4,
                                                                   reinterpret_cast<uint2*>(stage));
  RDM_LAUNCHED(ctx);
}

void widen_cols(rdm_ctx* ctx, const void* stage, int64_t n, int64_t ld, int64_t skip_lo, int64_t skip_hi,
                float* col) {
  const int64_t n4 = n * ld / 4;
  if (!n4) return;
  widen_cols_kernel<<<grid_for(ctx, n4), 256, 0, ctx->stream>>>(reinterpret_cast<const uint2*>(stage), n4,
                                                                  skip_lo * ld / 4, skip_hi * ld / 4, col);
  RDM_LAUNCHED(ctx);
}

namespace {
__global__ void scatter_kernel(const float* __restrict__ src, int64_t lds, int64_t rows, int64_t cols,
                               Scatter s) {
  const int64_t total = rows * cols;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / cols, c = i % cols;
    const float x = src[r * lds + c];
    if (s.mode == 1) {   // row slice → column slices (global rows my_off + r)
      int q = 0;
      while (q + 1 < s.P && s.lo[q + 1] <= c) ++q;
      s.ptr[q][(s.my_off + r) * s.ld[q] + (c - s.lo[q])] = x;
    } else if (c < s.my_w) {   // column slice → row slices (global columns my_off + c)
      int q = 0;
      while (q + 1 < s.P && s.lo[q + 1] <= r) ++q;
      s.ptr[q][(r - s.lo[q]) * s.ld[q] + s.my_off + c] = x;
    }
  }
}
}  // namespace

void scatter_slice(rdm_ctx* ctx, const float* src, int64_t lds, int64_t rows, int64_t cols,
                   const Scatter& s) {
  if (rows == 0 || cols == 0) return;
  scatter_kernel<<<grid_for(ctx, rows * cols), 256, 0, ctx->stream>>>(src, lds, rows, cols, s);
  RDM_LAUNCHED(ctx);
}

}  // namespace rdm
