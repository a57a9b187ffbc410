// misc.cu — loss, Hadamard mask, reductions, Adam, CSR validation.
//
//  * softmax cross-entropy ("the loss function typically needs
//    all the embeddings for a single vertex to be in the same process";
//    reading R5: mean over the train mask, global n_train) fused forward +
//    backward:  G^L = (softmax(Z^L) − onehot(y)) ⊙ m / n_train.
//  * Hadamard with σ'(Z) = 1[Z > 0] (eq. 3) when it cannot ride an epilogue.
//  * Adam (L297: lr 0.01; reading R10: PyTorch defaults).
// All reductions are fixed-order (deterministic), no float atomics.
#include <cfloat>

#include "internal.h"

namespace rdm {
namespace {

constexpr int kLossBlocks = 592;   // 4 x 148 SMs; fixed => deterministic partials
constexpr int kLossWarps = 8;

__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}
__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ double warp_sum_d(double v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// One warp per row (grid-stride with a fixed grid); block partial sums of the
// per-row losses in fp64 → partial[blockIdx.x].
__global__ void __launch_bounds__(kLossWarps * 32)
xent_kernel(const float* __restrict__ Z, int64_t ldz, const int32_t* __restrict__ labels,
            const uint8_t* __restrict__ mask, int64_t rows, int64_t C,
            const double* __restrict__ n_train, float* __restrict__ G, int64_t ldg,
            double* __restrict__ partial) {
  __shared__ double red[kLossWarps];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const double nt = *n_train;
  const float inv_n = nt > 0 ? (float)(1.0 / nt) : 0.f;
  double local = 0.0;
  constexpr int NV = 8;  // logits held in registers for C <= 256
  for (int64_t i = (int64_t)blockIdx.x * kLossWarps + wid; i < rows;
       i += (int64_t)gridDim.x * kLossWarps) {
    const float* z = Z + i * ldz;
    const int y = labels[i];
    const bool m = mask ? mask[i] != 0 : true;
    const float scale = m ? inv_n : 0.f;
    float* g = G + i * ldg;
    float mx = -FLT_MAX, s = 0.f, zy = 0.f;
    if (C <= 32 * NV) {
      float v[NV];
#pragma unroll
      for (int t = 0; t < NV; ++t) {
        const int64_t c = lane + 32 * t;
        v[t] = c < C ? z[c] : -FLT_MAX;
        mx = fmaxf(mx, v[t]);
      }
      mx = warp_max(mx);
#pragma unroll
      for (int t = 0; t < NV; ++t) {
        const int64_t c = lane + 32 * t;
        v[t] = c < C ? expf(v[t] - mx) : 0.f;
        s += v[t];
      }
      s = warp_sum(s);
      const float inv_s = 1.f / s;
#pragma unroll
      for (int t = 0; t < NV; ++t) {
        const int64_t c = lane + 32 * t;
        if (c < C) g[c] = (v[t] * inv_s - (c == y ? 1.f : 0.f)) * scale;
      }
    } else {
      for (int64_t c = lane; c < C; c += 32) mx = fmaxf(mx, z[c]);
      mx = warp_max(mx);
      for (int64_t c = lane; c < C; c += 32) s += expf(z[c] - mx);
      s = warp_sum(s);
      const float inv_s = 1.f / s;
      for (int64_t c = lane; c < C; c += 32) {
        const float p = expf(z[c] - mx) * inv_s;
        g[c] = (p - (c == y ? 1.f : 0.f)) * scale;
      }
    }
    if (lane == 0 && m) {
      zy = z[y];
      local += (double)mx + log((double)s) - (double)zy;
    }
  }
  if (lane == 0) red[wid] = local;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int k = 0; k < kLossWarps; ++k) t += red[k];
    partial[blockIdx.x] = t;
  }
}

// Narrow rows (C ≤ 128): LPR lanes per row, EPL = 4·V columns per lane as V
// float4 loads, 32/LPR rows per warp in flight (the one-warp-per-row kernel
// above serialises two full-warp reductions per row, latency-bound for
// C = 41 / 47).  Rows are 16-byte aligned with zero pads (executor layout);
// pads are excluded from the max / sum and written back as zeros.
template <int LPR, int V>
__global__ void __launch_bounds__(kLossWarps * 32)
xent_group_kernel(const float* __restrict__ Z, int64_t ldz, const int32_t* __restrict__ labels,
                  const uint8_t* __restrict__ mask, int64_t rows, int64_t C,
                  const double* __restrict__ n_train, float* __restrict__ G, int64_t ldg,
                  double* __restrict__ partial) {
  constexpr int RPW = 32 / LPR;
  __shared__ double red[kLossWarps];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int sub = lane % LPR, grp = lane / LPR;
  const double nt = *n_train;
  const float inv_n = nt > 0 ? (float)(1.0 / nt) : 0.f;
  double local = 0.0;
  const int64_t stride = (int64_t)gridDim.x * kLossWarps * RPW;
  for (int64_t base = ((int64_t)blockIdx.x * kLossWarps + wid) * RPW; base < rows; base += stride) {
    const int64_t i = base + grp;
    const bool valid = i < rows;
    // label and mask issued with the logits (no dependent load after the
    // reductions); the label's logit is picked from registers below
    const int y = valid ? __ldg(labels + i) : -1;
    const bool m = valid && (mask ? __ldg(mask + i) != 0 : true);
    float4 v[V];
    float mx = -FLT_MAX, zy = 0.f;
#pragma unroll
    for (int k = 0; k < V; ++k) {
      const int64_t c = 4 * (sub + LPR * k);
      v[k] = (valid && c < C) ? __ldcs(reinterpret_cast<const float4*>(Z + i * ldz + c))
                              : make_float4(-FLT_MAX, -FLT_MAX, -FLT_MAX, -FLT_MAX);
      if (c + 1 >= C) v[k].y = -FLT_MAX;
      if (c + 2 >= C) v[k].z = -FLT_MAX;
      if (c + 3 >= C) v[k].w = -FLT_MAX;
      mx = fmaxf(mx, fmaxf(fmaxf(v[k].x, v[k].y), fmaxf(v[k].z, v[k].w)));
      if (y == c) zy = v[k].x;
      if (y == c + 1) zy = v[k].y;
      if (y == c + 2) zy = v[k].z;
      if (y == c + 3) zy = v[k].w;
    }
    // exactly one lane of the group holds z_y: a sum of it and zeros is exact
#pragma unroll
    for (int o = LPR / 2; o; o >>= 1) zy += __shfl_xor_sync(0xffffffffu, zy, o);
#pragma unroll
    for (int o = LPR / 2; o; o >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    float s = 0.f;
#pragma unroll
    for (int k = 0; k < V; ++k) {
      v[k].x = expf(v[k].x - mx);   // exp(-FLT_MAX - mx) = 0 for pads
      v[k].y = expf(v[k].y - mx);
      v[k].z = expf(v[k].z - mx);
      v[k].w = expf(v[k].w - mx);
      s += (v[k].x + v[k].y) + (v[k].z + v[k].w);
    }
#pragma unroll
    for (int o = LPR / 2; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (valid) {
      const float scale = m ? inv_n : 0.f;
      const float inv_s = 1.f / s;
#pragma unroll
      for (int k = 0; k < V; ++k) {
        const int64_t c = 4 * (sub + LPR * k);
        if (c < C) {
          float4 gv;
          gv.x = (v[k].x * inv_s - (c == y ? 1.f : 0.f)) * scale;
          gv.y = c + 1 < C ? (v[k].y * inv_s - (c + 1 == y ? 1.f : 0.f)) * scale : 0.f;
          gv.z = c + 2 < C ? (v[k].z * inv_s - (c + 2 == y ? 1.f : 0.f)) * scale : 0.f;
          gv.w = c + 3 < C ? (v[k].w * inv_s - (c + 3 == y ? 1.f : 0.f)) * scale : 0.f;
          *reinterpret_cast<float4*>(G + i * ldg + c) = gv;
        }
      }
      if (sub == 0 && m) local += (double)mx + log((double)s) - (double)zy;
    }
  }
  local = warp_sum_d(local);
  if (lane == 0) red[wid] = local;
  __syncthreads();
  if (threadIdx.x == 0) {
    double t = 0.0;
    for (int k = 0; k < kLossWarps; ++k) t += red[k];
    partial[blockIdx.x] = t;
  }
}

// Single-block ordered sum of n doubles (fixed tree) → *out.
__global__ void sum_partials(const double* __restrict__ p, int n, double* __restrict__ out) {
  __shared__ double s[1024];
  double v = 0.0;
  for (int k = threadIdx.x; k < n; k += blockDim.x) v += p[k];
  s[threadIdx.x] = v;
  __syncthreads();
  for (int o = blockDim.x / 2; o; o >>= 1) {
    if ((int)threadIdx.x < o) s[threadIdx.x] += s[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) *out = s[0];
}

__global__ void mask_count_kernel(const uint8_t* __restrict__ mask, int64_t rows,
                                  double* __restrict__ partial) {
  __shared__ double red[256];
  double v = 0.0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < rows;
       i += (int64_t)gridDim.x * blockDim.x)
    v += mask ? (mask[i] ? 1.0 : 0.0) : 1.0;
  red[threadIdx.x] = v;
  __syncthreads();
  for (int o = blockDim.x / 2; o; o >>= 1) {
    if ((int)threadIdx.x < o) red[threadIdx.x] += red[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) partial[blockIdx.x] = red[0];
}

__global__ void apply_mask_kernel(float* __restrict__ X, int64_t ldx, const float* __restrict__ H,
                                  int64_t ldh, int64_t rows, int64_t cols4) {
  const int64_t total = rows * cols4;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total;
       g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = g / cols4, c = (g % cols4) * 4;
    float4* x = reinterpret_cast<float4*>(X + i * ldx + c);
    const float4 h = __ldg(reinterpret_cast<const float4*>(H + i * ldh + c));
    float4 v = *x;
    v.x = h.x > 0.f ? v.x : 0.f;
    v.y = h.y > 0.f ? v.y : 0.f;
    v.z = h.z > 0.f ? v.z : 0.f;
    v.w = h.w > 0.f ? v.w : 0.f;
    *x = v;
  }
}

// db^l = 1ᵀ G^l (reading R8), deterministic: CTA (column tile of 32, row
// chunk) — lane = column, warp w sums rows chunk_lo + w, + 8, … in fp64 (each
// warp load is one 128-byte row segment); the 8 warp sums are added in warp
// order and the chunk partials in chunk order by colsum_finish_kernel.
constexpr int kColsumRows = 512;   // rows per chunk
__global__ void __launch_bounds__(256) colsum_kernel(const float* __restrict__ G, int64_t ldg,
                                                     int64_t rows, int64_t cols, int64_t rows_per,
                                                     double* __restrict__ part) {
  __shared__ double red[8][33];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t c = (int64_t)blockIdx.x * 32 + lane;
  const int64_t r0 = (int64_t)blockIdx.y * rows_per, r1 = min(rows, r0 + rows_per);
  double s = 0.0;
  if (c < cols)
    for (int64_t r = r0 + warp; r < r1; r += 8) s += (double)__ldg(G + r * ldg + c);
  red[warp][lane] = s;
  __syncthreads();
  if (warp == 0) {
    double t = 0.0;
#pragma unroll
    for (int w = 0; w < 8; ++w) t += red[w][lane];
    if (c < cols) part[(int64_t)blockIdx.y * cols + c] = t;
  }
}

__global__ void colsum_finish_kernel(const double* __restrict__ part, int nchunks, int64_t cols,
                                     float* __restrict__ out) {
  const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= cols) return;
  double t = 0.0;
  for (int k = 0; k < nchunks; ++k) t += part[(int64_t)k * cols + c];
  out[c] = (float)t;
}

struct PtrTab {
  const float* p[BlockTable::kMax];
};
struct PtrTabD {
  const double* p[BlockTable::kMax];
};

__global__ void sum_slots_kernel(float* __restrict__ out, PtrTab t, int n, int64_t count) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
       i += (int64_t)gridDim.x * blockDim.x) {
    float s = 0.f;
    for (int k = 0; k < n; ++k) s += t.p[k][i];
    out[i] = s;
  }
}

__global__ void sum_doubles_kernel(double* __restrict__ out, PtrTabD t, int n) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    double s = 0.0;
    for (int k = 0; k < n; ++k) s += *t.p[k];
    *out = s;
  }
}

__global__ void finish_loss_kernel(const double* sum, const double* n_train, double* loss) {
  if (threadIdx.x == 0) *loss = *n_train > 0 ? *sum / *n_train : 0.0;
}

__global__ void adam_kernel(float* __restrict__ p, const float* __restrict__ g,
                            float* __restrict__ m, float* __restrict__ v, int64_t n, float lr,
                            float b1, float b2, float eps, float bc1, float bc2) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const float gi = g[i];
    const float mi = b1 * m[i] + (1.f - b1) * gi;
    const float vi = b2 * v[i] + (1.f - b2) * gi * gi;
    m[i] = mi;
    v[i] = vi;
    const float mhat = mi / bc1;
    const float vhat = vi / bc2;
    p[i] -= lr * mhat / (sqrtf(vhat) + eps);
  }
}

__global__ void validate_csr_kernel(const int64_t* __restrict__ rowptr,
                                    const int32_t* __restrict__ col, int64_t n, int64_t nnz,
                                    int* __restrict__ bad) {
  const int64_t lim = nnz > n ? nnz : n;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < lim;
       i += (int64_t)gridDim.x * blockDim.x) {
    if (i < nnz) {
      const int32_t c = col[i];
      if (c < 0 || (int64_t)c >= n) atomicOr(bad, 1);
    }
    if (i < n && rowptr[i + 1] < rowptr[i]) atomicOr(bad, 2);
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    if (rowptr[0] != 0 || rowptr[n] != nnz) atomicOr(bad, 4);
  }
}

unsigned grid_for(rdm_ctx* ctx, int64_t total, int per = 256) {
  const int64_t want = ceil_div(total, per);
  return (unsigned)std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)ctx->num_sms * 16));
}

}  // namespace

void softmax_xent(rdm_ctx* ctx, const float* Z, int64_t ldz, const int32_t* labels,
                  const uint8_t* mask, int64_t rows, int64_t C, const double* n_train, float* G,
                  int64_t ldg, double* loss_partial) {
  // ≈2 rows per warp; the grid depends only on `rows`, so the partials and
  // their ordered sum are deterministic
  const bool aligned = ldz % 4 == 0 && ldg % 4 == 0 && ((uintptr_t)Z & 15) == 0 && ((uintptr_t)G & 15) == 0;
  if (aligned && C <= 128) {
    // lanes per row: the fewest with ≤ 8 columns each (V ≤ 2 float4), ≥ 2
    int lpr = 2;
    while (lpr < 32 && lpr * 8 < C) lpr *= 2;
    const int V = (int)ceil_div(C, 4 * lpr);
    const int rpb = kLossWarps * (32 / lpr);
    const int nb = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(rows, rpb * 2), 16384));
    double* part = reinterpret_cast<double*>(ensure_ws(ctx->ws_scratch, (size_t)nb * sizeof(double)));
#define RDM_XENT_CASE(l_, v_)                                                                          \
  if (lpr == l_ && V == v_)                                                                          \
    xent_group_kernel<l_, v_><<<nb, kLossWarps * 32, 0, ctx->stream>>>(Z, ldz, labels, mask, rows, C, \
                                                                       n_train, G, ldg, part);       \
  else
    RDM_XENT_CASE(2, 1) RDM_XENT_CASE(2, 2) RDM_XENT_CASE(4, 1) RDM_XENT_CASE(4, 2)
    RDM_XENT_CASE(8, 1) RDM_XENT_CASE(8, 2) RDM_XENT_CASE(16, 1) RDM_XENT_CASE(16, 2)
    throw Error(RDM_ERR_STATE, "xent: no kernel for the row shape");
#undef RDM_XENT_CASE
    RDM_LAUNCHED(ctx);
    sum_partials<<<1, 1024, 0, ctx->stream>>>(part, nb, loss_partial);
    RDM_LAUNCHED(ctx);
    return;
  }
  const int nb = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(rows, kLossWarps * 2), 16384));
  double* part = reinterpret_cast<double*>(ensure_ws(ctx->ws_scratch, (size_t)nb * sizeof(double)));
  xent_kernel<<<nb, kLossWarps * 32, 0, ctx->stream>>>(Z, ldz, labels, mask, rows, C, n_train, G,
                                                       ldg, part);
  RDM_LAUNCHED(ctx);
  sum_partials<<<1, 1024, 0, ctx->stream>>>(part, nb, loss_partial);
  RDM_LAUNCHED(ctx);
}

void count_mask(rdm_ctx* ctx, const uint8_t* mask, int64_t rows, double* out) {
  double* part = reinterpret_cast<double*>(ensure_ws(ctx->ws_scratch, kLossBlocks * sizeof(double)));
  mask_count_kernel<<<kLossBlocks, 256, 0, ctx->stream>>>(mask, rows, part);
  RDM_LAUNCHED(ctx);
  sum_partials<<<1, 1024, 0, ctx->stream>>>(part, kLossBlocks, out);
  RDM_LAUNCHED(ctx);
}

void apply_mask(rdm_ctx* ctx, float* X, int64_t ldx, const float* H, int64_t ldh, int64_t rows,
                int64_t cols) {
  const int64_t c4 = roundup4(cols) / 4;
  if (rows * c4 == 0) return;
  apply_mask_kernel<<<grid_for(ctx, rows * c4), 256, 0, ctx->stream>>>(X, ldx, H, ldh, rows, c4);
  RDM_LAUNCHED(ctx);
}

void colsum(rdm_ctx* ctx, const float* G, int64_t ldg, int64_t rows, int64_t cols, float* out) {
  if (cols <= 0) return;
  const int64_t ct = (cols + 31) / 32;
  // ~4 CTAs per SM over the whole grid, chunks of at least kColsumRows rows
  const int64_t want = std::max<int64_t>(1, (int64_t)4 * ctx->num_sms / ct);
  const int64_t nchunks = std::max<int64_t>(1, std::min(want, ceil_div(rows, kColsumRows)));
  const int64_t rows_per = std::max<int64_t>(1, ceil_div(rows, nchunks));
  double* part = reinterpret_cast<double*>(ensure_ws(ctx->ws_scratch, (size_t)nchunks * cols * sizeof(double)));
  colsum_kernel<<<dim3((unsigned)ct, (unsigned)nchunks), 256, 0, ctx->stream>>>(G, ldg, rows, cols, rows_per, part);
  RDM_LAUNCHED(ctx);
  colsum_finish_kernel<<<(unsigned)ceil_div(cols, 128), 128, 0, ctx->stream>>>(part, (int)nchunks, cols, out);
  RDM_LAUNCHED(ctx);
}

void sum_slots(rdm_ctx* ctx, float* out, const float* const* parts, int nparts, int64_t count) {
  RDM_CHECK_ARG(nparts <= BlockTable::kMax, "too many slots");
  PtrTab t{};
  for (int k = 0; k < nparts; ++k) t.p[k] = parts[k];
  sum_slots_kernel<<<grid_for(ctx, count), 256, 0, ctx->stream>>>(out, t, nparts, count);
  RDM_LAUNCHED(ctx);
}

void sum_doubles(rdm_ctx* ctx, double* out, const double* const* parts, int nparts) {
  PtrTabD t{};
  for (int k = 0; k < nparts; ++k) t.p[k] = parts[k];
  sum_doubles_kernel<<<1, 32, 0, ctx->stream>>>(out, t, nparts);
  RDM_LAUNCHED(ctx);
}

void finish_loss(rdm_ctx* ctx, const double* sum, const double* n_train, double* loss) {
  finish_loss_kernel<<<1, 32, 0, ctx->stream>>>(sum, n_train, loss);
  RDM_LAUNCHED(ctx);
}

void adam(rdm_ctx* ctx, float* p, const float* g, float* m, float* v, int64_t n, float lr,
          float b1, float b2, float eps, float bc1, float bc2) {
  if (n == 0) return;
  adam_kernel<<<grid_for(ctx, n), 256, 0, ctx->stream>>>(p, g, m, v, n, lr, b1, b2, eps, bc1, bc2);
  RDM_LAUNCHED(ctx);
}

__global__ void copy_2d_kernel(float* __restrict__ dst, int64_t ldd, const float* __restrict__ src,
                               int64_t lds, int64_t rows, int64_t cols) {
  const int64_t total = rows * cols;
  for (int64_t g = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; g < total;
       g += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = g / cols, c = g % cols;
    dst[r * ldd + c] = src[r * lds + c];
  }
}

void copy_2d(rdm_ctx* ctx, float* dst, int64_t ldd, const float* src, int64_t lds, int64_t rows,
             int64_t cols) {
  if (rows * cols == 0) return;
  const int64_t want = ceil_div(rows * cols, 256);
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)ctx->num_sms * 16));
  copy_2d_kernel<<<grid, 256, 0, ctx->stream>>>(dst, ldd, src, lds, rows, cols);
  RDM_LAUNCHED(ctx);
}

int validate_csr(rdm_ctx* ctx, const int64_t* rowptr, const int32_t* col, int64_t n, int64_t nnz) {
  int* flag = reinterpret_cast<int*>(ensure_ws(ctx->ws_scratch, 64));
  RDM_CUDA(cudaMemsetAsync(flag, 0, sizeof(int), ctx->stream));
  validate_csr_kernel<<<grid_for(ctx, std::max<int64_t>(nnz, n)), 256, 0, ctx->stream>>>(
      rowptr, col, n, nnz, flag);
  RDM_LAUNCHED(ctx);
  int h = 0;
  RDM_CUDA(cudaMemcpyAsync(&h, flag, sizeof(int), cudaMemcpyDeviceToHost, ctx->stream));
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  return h;
}

}  // namespace rdm
