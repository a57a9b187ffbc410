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
