// gemm_simt.cu — fp32 SIMT GEMM (CUDA cores) for the communication-free
// row-sliced products of the GCN layer (Fig. 2b):
//   NN  C = X · W        (eq. 1: Z = T W or T = H W)
//   NT  C = X · Wᵀ       (eq. 3: A G Wᵀ)
//   TN  C = Xᵀ · U       (eq. 4: Y = Hᵀ (A G)), split-K over rows with a
//                         deterministic ordered reduction (no float atomics).
// This is the portable fallback-free baseline used for shapes the tcgen05
// kernel (gemm_tc.cu) does not take; both are exact-fp32-class.
#include <algorithm>

#include "internal.h"

namespace rdm {
namespace {

constexpr int BM = 64, BN = 64, BK = 16, NT = 256;

struct GemmEpi {
  int flags;
  const float* bias;
  const float* mask;
  int64_t ld_mask;
};

// A(i, kk) = a_kmajor ? A[i*lda + kk] : A[kk*lda + i]
// B(kk, n) = b_nmajor ? B[kk*ldb + n] : B[n*ldb + kk]
template <bool A_KMAJOR, bool B_NMAJOR>
__global__ void __launch_bounds__(NT)
gemm_simt_kernel(const float* __restrict__ A, int64_t lda, const float* __restrict__ B, int64_t ldb,
                 float* __restrict__ C, int64_t ldc, int64_t M, int64_t N, int64_t K,
                 int64_t k_per_split, GemmEpi epi) {
  __shared__ float As[BK][BM + 4];
  __shared__ float Bs[BK][BN + 4];
  const int t = threadIdx.x;
  const int tx = t % 16, ty = t / 16;
  const int64_t m0 = (int64_t)blockIdx.x * BM, n0 = (int64_t)blockIdx.y * BN;
  const int64_t kbeg = (int64_t)blockIdx.z * k_per_split;
  const int64_t kend = min(K, kbeg + k_per_split);
  float acc[4][4] = {};
  for (int64_t k0 = kbeg; k0 < kend; k0 += BK) {
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      int i, kk;
      if (A_KMAJOR) { i = t / 4; kk = (t % 4) * 4 + e; }
      else          { kk = t / 16; i = (t % 16) * 4 + e; }
      const int64_t gi = m0 + i, gk = k0 + kk;
      float v = 0.f;
      if (gi < M && gk < kend) v = A_KMAJOR ? A[gi * lda + gk] : A[gk * lda + gi];
      As[kk][i] = v;
      int n, kb;
      if (B_NMAJOR) { kb = t / 16; n = (t % 16) * 4 + e; }
      else          { n = t / 4; kb = (t % 4) * 4 + e; }
      const int64_t gn = n0 + n, gkb = k0 + kb;
      float u = 0.f;
      if (gn < N && gkb < kend) u = B_NMAJOR ? B[gkb * ldb + gn] : B[gn * ldb + gkb];
      Bs[kb][n] = u;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int x = 0; x < 4; ++x) a[x] = As[kk][ty * 4 + x];
#pragma unroll
      for (int y = 0; y < 4; ++y) b[y] = Bs[kk][tx * 4 + y];
#pragma unroll
      for (int x = 0; x < 4; ++x)
#pragma unroll
        for (int y = 0; y < 4; ++y) acc[x][y] = fmaf(a[x], b[y], acc[x][y]);
    }
    __syncthreads();
  }
  // C is either the final output (gridDim.z == 1) or split-partial slab z
  float* Cz = C + (int64_t)blockIdx.z * M * ldc;
#pragma unroll
  for (int x = 0; x < 4; ++x) {
    const int64_t gi = m0 + ty * 4 + x;
    if (gi >= M) continue;
#pragma unroll
    for (int y = 0; y < 4; ++y) {
      const int64_t gn = n0 + tx * 4 + y;
      if (gn >= N) continue;
      float v = acc[x][y];
      if (gridDim.z == 1) {
        if (epi.flags & RDM_EPI_BIAS) v += epi.bias[gn];
        if (epi.flags & RDM_EPI_RELU) v = fmaxf(v, 0.f);
        if ((epi.flags & RDM_EPI_MASK) && !(epi.mask[gi * epi.ld_mask + gn] > 0.f)) v = 0.f;
      }
      Cz[gi * ldc + gn] = v;
    }
  }
}

// Ordered sum of split-K partial slabs (deterministic).
__global__ void splitk_reduce(const float* __restrict__ part, int splits, int64_t M, int64_t N,
                              float* __restrict__ C, int64_t ldc) {
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= M * N) return;
  const int64_t i = idx / N, n = idx % N;
  float s = 0.f;
  for (int z = 0; z < splits; ++z) s += part[(int64_t)z * M * N + i * N + n];
  C[i * ldc + n] = s;
}

template <bool AK, bool BNm>
void launch(rdm_ctx* ctx, const float* A, int64_t lda, const float* B, int64_t ldb, float* C,
            int64_t ldc, int64_t M, int64_t N, int64_t K, int splits, const GemmEpi& e) {
  const int64_t kps = ceil_div(ceil_div(K, splits), BK) * BK;
  dim3 grid((unsigned)ceil_div(M, BM), (unsigned)ceil_div(N, BN), (unsigned)splits);
  gemm_simt_kernel<AK, BNm><<<grid, NT, 0, ctx->stream>>>(A, lda, B, ldb, C, ldc, M, N, K, kps, e);
  RDM_LAUNCHED(ctx);
}

}  // namespace

void gemm_simt(rdm_ctx* ctx, int op, const float* X, int64_t ldx, const float* W, int64_t ldw,
               float* C, int64_t ldc, int64_t rows, int64_t k, int64_t m, int epi_flags,
               const float* bias, const float* mask) {
  GemmEpi e{epi_flags, bias, mask, ldc};
  if (op == RDM_GEMM_NN) {
    launch<true, true>(ctx, X, ldx, W, ldw, C, ldc, rows, m, k, 1, e);
  } else if (op == RDM_GEMM_NT) {
    launch<true, false>(ctx, X, ldx, W, ldw, C, ldc, rows, k, m, 1, e);
  } else {
    // TN: C[k x m] = Xᵀ U, K = rows (huge): split-K
    const int64_t tiles = ceil_div(k, BM) * ceil_div(m, BN);
    int64_t splits = std::max<int64_t>(1, (4 * ctx->num_sms) / std::max<int64_t>(1, tiles));
    splits = std::min<int64_t>(splits, std::max<int64_t>(1, rows / 512));
    splits = std::min<int64_t>(splits, 1024);
    if (splits == 1) {
      launch<false, true>(ctx, X, ldx, W, ldw, C, ldc, k, m, rows, 1, GemmEpi{0, nullptr, nullptr, 0});
    } else {
      float* part = ensure_ws(ctx->ws_gemm, (size_t)splits * k * m * sizeof(float));
      launch<false, true>(ctx, X, ldx, W, ldw, part, m, k, m, rows, (int)splits,
                          GemmEpi{0, nullptr, nullptr, 0});
      const int64_t tot = k * m;
      splitk_reduce<<<(unsigned)ceil_div(tot, 256), 256, 0, ctx->stream>>>(part, (int)splits, k, m,
                                                                           C, ldc);
      RDM_LAUNCHED(ctx);
    }
  }
}

}  // namespace rdm
