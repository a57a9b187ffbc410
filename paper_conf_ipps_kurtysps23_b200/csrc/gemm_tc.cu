// gemm_tc.cu — fp32-accurate GEMM on the 5th-generation tensor cores (sm_100a).
//
// The communication-free dense products of the GCN layer (Fig. 2b,
// L112: W replicated, row-sliced operands) — eq. (1) Z = T·W, eq. (3) A·G·Wᵀ,
// eq. (4) Y = Hᵀ·(A·G) — run as tcgen05.mma kind::tf32 with the 3xTF32 split
// (x = hi + lo, hi = x with the 13 low mantissa bits cleared, lo = x − hi
// exactly; C = A_hi·B_hi + A_hi·B_lo + A_lo·B_hi), which keeps fp32-class
// accuracy (the 1e-4 parity gate excludes 1xTF32's 2^-11 unit roundoff).
//
// Per CTA: one 128 x BN output tile accumulated in TMEM (fp32).  Warp roles:
//   warp 0  TMA producer (cp.async.bulk.tensor, 128B swizzle, mbarrier tx)
//   warp 1  MMA issuer (one thread issues tcgen05.mma; tcgen05.commit frees
//           the smem stage and finally signals the epilogue)
//   warp 2  TMEM allocator
//   warps 4-7  split converter (in-place hi, lo into a twin buffer, then
//           fence.proxy.async so the tensor core sees it) and afterwards the
//           epilogue (tcgen05.ld 32x32b → fused ReLU / Hadamard mask / bias →
//           global), one TMEM lane quadrant per warp.
// Modes:
//   NN / NT  A = X (K-major, TMA box 32 x 128); B = W or Wᵀ pre-split into
//            hi/lo K-major panels by a tiny prep kernel (W is ≤ 1433 x 256).
//   TN       A = Xᵀ and B = U are MN-major in memory (rows of X / U are the
//            contraction): both loaded MN-major (box 32 x 32 per 128-byte
//            chunk) with MN-major UMMA descriptors, both split in smem;
//            split-K over rows with an ordered (deterministic) reduction.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_bf16.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "internal.h"
#include "tc_ptx.h"

namespace rdm {
namespace {
using namespace tc;

constexpr int BK = 32;         // fp32 elements per 128-byte swizzle row

// Timeline trace of CTA 0 (build with -DRDM_TC_TRACE, tools/build_variant.sh;
// read with rdm_debug_tc_trace, tools/tc_trace.py): clock64 per role and
// k-block / tile.
#ifdef RDM_TC_TRACE
constexpr int kTrN = 4096;
__device__ long long g_tc_trace[8][kTrN];
#define TCTRACE(ev, idx)                                                        \
  do {                                                                          \
    if (blockIdx.x == 0 && (idx) < kTrN) g_tc_trace[ev][idx] = clock64();      \
  } while (0)
#else
#define TCTRACE(ev, idx) do { } while (0)
#endif
constexpr int UK = 8;          // UMMA K for kind::tf32

struct TcEpi {
  int flags;
  const float* bias;
  const float* mask;
  int64_t ld_mask;
  Scatter scat;   // fused row→column redistribution (MODE 0, no split-K); scat.P == 0: off
  // RDM_PREC_FAST: a bf16 copy of the output (× twin_scale[row] when not null),
  // row length ld_twin, columns [N, ld_twin) zero — the next SpMM's input
  // (the cast folded into this epilogue); null: off
  uint16_t* twin = nullptr;
  int64_t ld_twin = 0;
  const float* twin_scale = nullptr;
  // ReLU sign bits of the output (1[v > 0], one u32 per 32 columns, row length
  // ld_bits_out words) for a later Hadamard; and the Hadamard read from such
  // bits instead of the fp32 mask (1/32 of its bytes)
  uint32_t* bits_out = nullptr;
  int64_t ld_bits_out = 0;
  const uint32_t* mask_bits = nullptr;
  int64_t ld_mask_bits = 0;
};

struct TcShape {
  int64_t M, N, K, k_per_split;
  int tiles_m, tiles_n, splits, n_mma;
  int pf;   // issue L2 prefetches of A through tmApf
  int dbg;  // timing experiments only (RDM_TC_DBG): 1 = skip split, 2 = skip MMA, 4 = skip stores
  int one;  // RDM_PREC_FAST: 1xTF32 (one MMA per k step, no lo operands)
  int tstore;  // epilogue stores through TMA (tmC) — MODE 0, one split, no fused scatter
};

// A operand placement.  For BN ≤ 128 the converter writes A's hi / lo split
// straight into TMEM (tcgen05.st) and the MMA reads A from TMEM: the smem
// stage then only carries the raw A tile and the B panels, which removes the
// smem-bandwidth bound of the converter (write hi + lo) plus three MMA reads
// of A per k-block.  BN = 256 needs all 512 TMEM columns for the two
// accumulators and keeps A in shared memory.
// EW = epilogue warps: 4 (one per TMEM lane quadrant) for mainloop-bound
// calls, 8 (two per quadrant, column halves) for epilogue-bound ones (short
// K, wide outputs) — 8 warps cost one smem stage of transpose buffers.
// PAIR = 2: a CTA pair (cluster of 2, tcgen05 cta_group::2) computes a
// 256 x BN tile: each CTA holds its own 128 rows of A and HALF of the B panel
// (BN/2 rows), the leader's MMAs (M = 256) read both halves, so every SM loads
// half the W panel bytes per row it computes.
// ASM = 1 (pairs, BN <= 128): A split in shared memory instead of TMEM, which
// leaves TMEM to two partial accumulators per buffer (the three MMAs of a k
// step alternate between them instead of serialising on one).
// F16 = 1 (fast variant, A in TMEM): kind::f16 MMAs on bf16 operands — A
// rounded to bf16 pairs by the converter (16 TMEM columns per 32-wide k-block),
// W as bf16 K-major panels with the 64-byte swizzle (64 B per row per k-block).
template <int BN, int EW, int PAIR = 1, int ASM = 0, int F16 = 0>
struct Cfg {
  static constexpr int kThreads = 256 + 32 * EW;
  static constexpr int kAccCols = BN <= 32 ? 32 : BN <= 64 ? 64 : BN <= 128 ? 128 : 256;
  static constexpr bool kTmemA = BN <= 128 && !ASM;
  // partial accumulators (the bf16 path issues 2 MMAs per k-block: at most 2)
  static constexpr int kNAcc = !kTmemA ? (BN <= 128 ? 2 : 1) : BN <= 32 ? (F16 ? 2 : 4) : BN <= 64 ? 2 : 1;
  static constexpr int kABytes = BM * BK * 4;   // 16 KB
  static constexpr int kBBytes = (BN / PAIR) * BK * (F16 ? 2 : 4);
  static constexpr int kStageBytes = (kTmemA ? 1 : 2) * kABytes + 2 * kBBytes;
  // per epilogue warp 5 KB (1024-aligned): a 32 x 33 transpose tile, or the
  // 32 x 32 swizzled box of a TMA store
  static constexpr int kEpiBytes = EW * 5120;
  static constexpr int kBudget = 224 * 1024 - kEpiBytes - 1024 - 512;
  // deep rings hide TMA latency.  With A in TMEM the converted A stages form
  // a second ring (64 TMEM columns each, whatever the accumulators leave),
  // decoupled from the smem ring of raw A + B tiles, which can run deeper.
  static constexpr int kAStride = F16 ? BK / 2 : 2 * BK;   // TMEM columns per A stage
  static constexpr int kStagesT0 = kTmemA ? (512 - 2 * kNAcc * kAccCols) / kAStride : 0;
  static constexpr int kStagesT = kStagesT0 < 8 ? kStagesT0 : 8;
  static constexpr int kMaxStages = kTmemA ? 8 : 4;
  static constexpr int kFitStages = kBudget / kStageBytes < 8 ? kBudget / kStageBytes : 8;
  static constexpr int kStages = kFitStages < kMaxStages ? kFitStages : kMaxStages;
  static constexpr int kSmem = kStages * kStageBytes + kEpiBytes + 1024 /*align*/ + 512 /*barriers*/;
  static constexpr int kACol0 = 2 * kNAcc * kAccCols;  // first TMEM column of the A stages
  static constexpr int kUsedCols = kACol0 + kStagesT * kAStride;
  static constexpr int kTmemCols = kUsedCols <= 32 ? 32 : kUsedCols <= 64 ? 64 : kUsedCols <= 128 ? 128
                                   : kUsedCols <= 256 ? 256 : 512;
  static_assert(kUsedCols <= 512, "TMEM overflow");
};

__device__ __forceinline__ void tc_mma_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db,
                                          uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate)
      : "memory");
}

template <int PAIR>
__device__ __forceinline__ void tc_mma_ts_g(uint32_t tmem_d, uint32_t tmem_a, uint64_t db,
                                            uint32_t idesc, uint32_t accumulate) {
  if (PAIR == 1) {
    tc_mma_ts(tmem_d, tmem_a, db, idesc, accumulate);
  } else {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::tf32 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
        "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate)
        : "memory");
  }
}
template <int PAIR>
__device__ __forceinline__ void tc_mma_g(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc,
                                         uint32_t accumulate) {
  if (PAIR == 1) {
    tc_mma(tmem_d, da, db, idesc, accumulate);
  } else {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(da), "l"(db), "r"(idesc), "r"(accumulate)
        : "memory");
  }
}
// kind::f16 (bf16) MMA with A from TMEM (bf16 pairs packed in 32-bit columns)
__device__ __forceinline__ void tc_mma_bf16_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t idesc,
                                               uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate)
      : "memory");
}
// kind::f16 instruction descriptor: D f32, A/B bf16, both K-major, M = 128, N.
__host__ __device__ constexpr uint32_t idesc_bf16k(int N) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}
__device__ __forceinline__ void tmem_st16u(uint32_t addr, const uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
          addr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]),
      "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
      : "memory");
}

template <int PAIR>
__device__ __forceinline__ void tc_commit_g(uint64_t* b) {
  if (PAIR == 1) tc_commit(b);
  else tc_commit_pair(b);
}

__device__ __forceinline__ void tmem_st32(uint32_t addr, const float (&v)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,"
      "%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(addr),
      "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]),
      "f"(v[8]), "f"(v[9]), "f"(v[10]), "f"(v[11]), "f"(v[12]), "f"(v[13]), "f"(v[14]), "f"(v[15]),
      "f"(v[16]), "f"(v[17]), "f"(v[18]), "f"(v[19]), "f"(v[20]), "f"(v[21]), "f"(v[22]), "f"(v[23]),
      "f"(v[24]), "f"(v[25]), "f"(v[26]), "f"(v[27]), "f"(v[28]), "f"(v[29]), "f"(v[30]), "f"(v[31])
      : "memory");
}

// Row m (0..127) of the raw A tile, 32 K values, from the swizzled smem stage.
//  MODE 0 (K-major, 128B swizzle): row m is the 128-byte line m, 16-byte chunk c
//          stored at chunk c ^ (m & 7).
//  MODE 1 (MN-major, 128B swizzle with 32-byte atoms): element (k, m) lives in
//          MN chunk m/32 (4 KB), line k, 32-byte atom ((m%32)/8) ^ (k & 3).
template <int MODE>
__device__ __forceinline__ void load_a_row(const uint8_t* tile, int m, float (&v)[32]) {
  if (MODE == 0) {
    const float4* line = reinterpret_cast<const float4*>(tile + m * 128);
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      const float4 x = line[c ^ (m & 7)];
      v[4 * c + 0] = x.x; v[4 * c + 1] = x.y; v[4 * c + 2] = x.z; v[4 * c + 3] = x.w;
    }
  } else {
    const uint8_t* chunk = tile + (m >> 5) * 4096;
    const int mm = m & 31;
#pragma unroll
    for (int k = 0; k < 32; ++k)
      v[k] = *reinterpret_cast<const float*>(chunk + k * 128 + ((((mm >> 3) ^ (k & 3)) << 5) | ((mm & 7) << 2)));
  }
}

// Persistent, warp-specialised tcgen05 GEMM.  384 threads:
//   warp 0      TMA producer           warp 1  MMA issuer (one thread)
//   warp 2      TMEM allocator         warp 3  idle
//   warps 4-7   3xTF32 split converter (in-place hi, lo twin buffer)
//   warps 8-11  epilogue: TMEM → registers → smem transpose → coalesced
//               global stores with fused bias / ReLU / Hadamard mask
// Tiles (m, n, split) are strided over the grid; the smem ring runs across
// tiles and the TMEM accumulator is double-buffered, so the epilogue of tile i
// overlaps the mainloop of tile i + 1.
// MODE 0: NN/NT (A K-major + converter, B pre-split K-major).
// MODE 1: TN (A, B MN-major, both split in smem), split-K slabs.
template <int BN, int MODE, int EW, int PAIR, int ASM, int F16>
__global__ void __launch_bounds__(256 + 32 * EW, 1)
gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
               const __grid_constant__ CUtensorMap tmBlo, const __grid_constant__ CUtensorMap tmApf,
               const __grid_constant__ CUtensorMap tmC, float* __restrict__ C, int64_t ldc,
               TcShape sh, TcEpi epi) {
  // (CTA pairs: NN / NT, and TN with MN-major B halves of 32-wide chunks)
  static_assert(!F16 || (MODE == 0 && PAIR == 1 && BN <= 128 && !ASM), "bf16 GEMM: NN / NT, A in TMEM");
  using CF = Cfg<BN, EW, PAIR, ASM, F16>;
  constexpr int S = CF::kStages;      // smem ring (raw A + B panels)
  constexpr int ST = CF::kStagesT;    // TMEM ring of converted A (kTmemA)
  constexpr int SC = CF::kTmemA ? ST : S;   // ring the converter hands to the MMA
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  uint8_t* stage_base = smem;
  float* epi_smem = (float*)(smem + S * CF::kStageBytes);
  uint64_t* full = (uint64_t*)(smem + S * CF::kStageBytes + CF::kEpiBytes);
  uint64_t* conv = full + S;     // [SC]
  uint64_t* empty = conv + SC;
  uint64_t* tfull = empty + S;   // [2]
  uint64_t* tempty = tfull + 2;  // [2]
  uint64_t* aempty = tempty + 2;  // [ST] TMEM A stage consumed by the MMAs
  uint32_t* tmem_slot = (uint32_t*)(aempty + (ST > 0 ? ST : 1));

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int tiles_mn = sh.tiles_m * sh.tiles_n;
  const int total = tiles_mn * sh.splits;
  // tiles are strided over CTAs (PAIR = 1) or CTA pairs (PAIR = 2: the two
  // CTAs of a cluster take the same tile, rows rank·128 … of its 256)
  const uint32_t rank = PAIR == 2 ? cluster_ctarank() : 0u;
  const int cta0 = PAIR == 2 ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
  const int ncta = PAIR == 2 ? (int)(gridDim.x >> 1) : (int)gridDim.x;
  // pair: the B half of this CTA (rows of the MMA's N) and its size in bytes
  const int b_rows = PAIR == 2 ? sh.n_mma / 2 : BN;

  constexpr int kAB = (CF::kTmemA ? 1 : 2) * CF::kABytes;   // A bytes per stage in smem
  auto A_hi = [&](int s) { return stage_base + s * CF::kStageBytes; };
  auto A_lo = [&](int s) { return stage_base + s * CF::kStageBytes + CF::kABytes; };  // !kTmemA only
  auto B_hi = [&](int s) { return stage_base + s * CF::kStageBytes + kAB; };
  auto B_lo = [&](int s) { return stage_base + s * CF::kStageBytes + kAB + CF::kBBytes; };
  auto tile_kb = [&](int t, int64_t& kbeg) {
    const int z = t / tiles_mn;
    kbeg = (int64_t)z * sh.k_per_split;
    const int64_t kend = min(sh.K, kbeg + sh.k_per_split);
    return kend > kbeg ? (int)((kend - kbeg + BK - 1) / BK) : 0;
  };

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    // pair: one arrival per converter warp of both CTAs, on the leader's barrier
    for (int s = 0; s < SC; ++s) mbar_init(&conv[s], PAIR == 2 ? 8 : 128);
    for (int s = 0; s < ST; ++s) mbar_init(&aempty[s], 1);
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull[b], 1);
      mbar_init(&tempty[b], PAIR == 2 ? 2 * EW : 32 * EW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 2) {
    if (PAIR == 2) {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                       smem_u32(tmem_slot)),
                   "n"(CF::kTmemCols));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    } else {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                       smem_u32(tmem_slot)),
                   "n"(CF::kTmemCols));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
  }
  tc_fence_before();
  __syncthreads();
  if (PAIR == 2) cluster_sync_all();   // both CTAs' barriers initialised before any remote arrival
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      const uint32_t bbytes = (uint32_t)b_rows * BK * (F16 ? 2 : 4);
      const uint32_t bytes = MODE == 0 ? (CF::kABytes + (sh.one ? 1 : 2) * bbytes) : (CF::kABytes + bbytes);
      uint32_t kc = 0;
      for (int t = cta0; t < total; t += ncta) {
        int64_t kbeg;
        const int nkb = tile_kb(t, kbeg);
        const int rem = t % tiles_mn;
        const int m0 = (rem / sh.tiles_n) * (BM * PAIR) + (int)rank * BM;
        const int n0 = (rem % sh.tiles_n) * BN + (int)rank * b_rows;
        for (int kb = 0; kb < nkb; ++kb, ++kc) {
          const int s = kc % S;
          if (kc >= (uint32_t)S) mbar_wait(&empty[s], ((kc / S) - 1) & 1);
          TCTRACE(0, kc);
          mbar_expect_tx(&full[s], bytes);
          const int kk = (int)(kbeg + (int64_t)kb * BK);
          if (MODE == 0) {
            // L2 prefetch of A in 512-byte row segments, one group (4 k-blocks)
            // ahead: the 128-byte swizzled boxes alone touch each DRAM page once
            // per k-block across thousands of concurrent rows.
            if (sh.pf) {
              const int g = kb >> 2;
              if ((kb & 3) == 0) {
                if (kb == 0) tma_prefetch_2d(&tmApf, kk, m0);
                if ((int64_t)(g + 1) * 4 < nkb) tma_prefetch_2d(&tmApf, kk + 4 * BK, m0);
              }
            }
            tma_load_2d(A_hi(s), &tmA, &full[s], kk, m0);
            tma_load_2d(B_hi(s), &tmB, &full[s], kk, n0);
            if (!sh.one) tma_load_2d(B_lo(s), &tmBlo, &full[s], kk, n0);
          } else {
            for (int c = 0; c < BM / 32; ++c) tma_load_2d(A_hi(s) + c * 4096, &tmA, &full[s], m0 + 32 * c, kk);
            for (int c = 0; c < b_rows / 32; ++c) tma_load_2d(B_hi(s) + c * 4096, &tmB, &full[s], n0 + 32 * c, kk);
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {   // pair: the leader CTA issues the pair's MMAs
      // A read from TMEM is K-major by construction (the converter writes rows)
      const uint32_t idesc = F16 ? idesc_bf16k(sh.n_mma) : idesc_tf32(sh.n_mma, CF::kTmemA ? 0 : MODE, MODE, BM * PAIR);
      uint32_t kc = 0;
      int it = 0;
      for (int t = cta0; t < total; t += ncta, ++it) {
        int64_t kbeg;
        const int nkb = tile_kb(t, kbeg);
        const int acc = it & 1;
        if (it >= 2) {
          if (PAIR == 2) mbar_wait_cluster(&tempty[acc], ((it >> 1) - 1) & 1);
          else mbar_wait(&tempty[acc], ((it >> 1) - 1) & 1);
        }
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * (CF::kNAcc * CF::kAccCols);
        for (int kb = 0; kb < nkb; ++kb, ++kc) {
          const int s = kc % S;
          const int st = CF::kTmemA ? (int)(kc % ST) : 0;
          const int cs = kc % SC;
          if (PAIR == 2) mbar_wait_cluster(&conv[cs], (kc / SC) & 1);
          else mbar_wait(&conv[cs], (kc / SC) & 1);
          TCTRACE(3, kc);
          tc_fence_after();
          const uint32_t bh = smem_u32(B_hi(s)), bl = smem_u32(B_lo(s));
          if (F16) {
            // two K = 16 steps per 32-wide k-block: 8 packed A columns and 32 B
            // of each 64-byte-swizzled B row per step
#pragma unroll
            for (int j = 0; j < 2; ++j) {
              const uint32_t d = d_tmem + (uint32_t)((j % CF::kNAcc) * CF::kAccCols);
              if (!(sh.dbg & 2))
                tc_mma_bf16_ts(d, tmem_base + CF::kACol0 + st * CF::kAStride + j * 8, sdesc(bh + j * 32, 16, 512, 4),
                               idesc, (kb > 0 || j >= CF::kNAcc) ? 1u : 0u);
            }
          }
#pragma unroll
          for (int j = 0; j < (F16 ? 0 : BK / UK); ++j) {
            uint64_t dbh, dbl;
            if (MODE == 0) {  // K-major: advance 32 B along the swizzled row
              dbh = sdesc(bh + j * 32, 16, 1024);
              dbl = sdesc(bl + j * 32, 16, 1024);
            } else {
              // MN-major tf32 needs the 128B swizzle with 32-byte atoms: K rows are
              // 128-byte lines, 4-row groups 512 B apart (SBO), 32-wide MN chunks
              // 4 KB apart (LBO); one K = 8 step spans two groups (1 KB).
              dbh = sdesc(bh + j * 1024, 4096, 512, 1);
              dbl = sdesc(bl + j * 1024, 4096, 512, 1);
            }
            const uint32_t acc0 = (kb > 0 || j > 0) ? 1u : 0u;
            if (sh.dbg & 2) {
            } else if (sh.one) {
              // 1xTF32: A_tf32 · B_tf32, rotating over the partial accumulators
              const uint32_t d = d_tmem + (uint32_t)((j % CF::kNAcc) * CF::kAccCols);
              if (CF::kTmemA) {
                tc_mma_ts_g<PAIR>(d, tmem_base + CF::kACol0 + st * CF::kAStride + j * UK, dbh, idesc,
                                  (kb > 0 || j >= CF::kNAcc) ? 1u : 0u);
              } else {
                const uint32_t ah = smem_u32(A_hi(s));
                tc_mma_g<PAIR>(d, MODE == 0 ? sdesc(ah + j * 32, 16, 1024) : sdesc(ah + j * 1024, 4096, 512, 1),
                               dbh, idesc, (kb > 0 || j >= CF::kNAcc) ? 1u : 0u);
              }
            } else if (CF::kTmemA) {
              // A stage st: hi in columns [kACol0 + 64 st, +32), lo in the next 32.
              // Narrow tiles rotate over kNAcc independent accumulators so that
              // consecutive MMAs do not serialise on one accumulator.
              const uint32_t ta = tmem_base + CF::kACol0 + st * CF::kAStride + j * UK;
              const uint32_t tab[3] = {ta, ta, ta + BK};
#pragma unroll
              for (int p = 0; p < 3; ++p) {
                const int i = j * 3 + p;
                const uint32_t d = d_tmem + (uint32_t)((i % CF::kNAcc) * CF::kAccCols);
                tc_mma_ts_g<PAIR>(d, tab[p], p == 1 ? dbl : dbh, idesc, (kb > 0 || i >= CF::kNAcc) ? 1u : 0u);
              }
            } else {
              const uint32_t ah = smem_u32(A_hi(s)), al = smem_u32(A_lo(s));
              uint64_t dah, dal;
              if (MODE == 0) {
                dah = sdesc(ah + j * 32, 16, 1024);
                dal = sdesc(al + j * 32, 16, 1024);
              } else {
                dah = sdesc(ah + j * 1024, 4096, 512, 1);
                dal = sdesc(al + j * 1024, 4096, 512, 1);
              }
              if (CF::kNAcc == 1) {
                tc_mma_g<PAIR>(d_tmem, dah, dbh, idesc, acc0);
                tc_mma_g<PAIR>(d_tmem, dah, dbl, idesc, 1u);
                tc_mma_g<PAIR>(d_tmem, dal, dbh, idesc, 1u);
              } else {
                const uint64_t da3[3] = {dah, dah, dal}, db3[3] = {dbh, dbl, dbh};
#pragma unroll
                for (int p = 0; p < 3; ++p) {
                  const int i = j * 3 + p;
                  const uint32_t d = d_tmem + (uint32_t)((i % CF::kNAcc) * CF::kAccCols);
                  tc_mma_g<PAIR>(d, da3[p], db3[p], idesc, (kb > 0 || i >= CF::kNAcc) ? 1u : 0u);
                }
              }
            }
          }
          tc_commit_g<PAIR>(&empty[s]);   // pair: frees the stage in both CTAs
          if (CF::kTmemA) tc_commit_g<PAIR>(&aempty[st]);
        }
        tc_commit_g<PAIR>(&tfull[acc]);   // fires when this tile's MMAs (if any) are done
        TCTRACE(4, it);
      }
    }
  } else if (warp >= 4 && warp < 8) {
    const int t128 = threadIdx.x - 128;
    const uint32_t conv_leader = PAIR == 2 ? mapa_u32(smem_u32(conv), 0) : 0u;
    uint32_t kc = 0;
    for (int t = cta0; t < total; t += ncta) {
      int64_t kbeg;
      const int nkb = tile_kb(t, kbeg);
      for (int kb = 0; kb < nkb; ++kb, ++kc) {
        const int s = kc % S;
        const int st = CF::kTmemA ? (int)(kc % ST) : 0;
        const int cs = kc % SC;
        if (CF::kTmemA && kc >= (uint32_t)ST) {   // the MMAs have read TMEM stage st
          mbar_wait(&aempty[st], ((kc / ST) - 1) & 1);
          tc_fence_after();
        }
        mbar_wait(&full[s], (kc / S) & 1);
        if (threadIdx.x == 128) TCTRACE(1, kc);
        if (sh.dbg & 1) {
        } else if (sh.one) {
          // 1xTF32: A rounded to tf32 into TMEM; smem operands are read as tf32
          // by the tensor core as they are (low mantissa bits ignored)
          if (CF::kTmemA && F16) {
            // bf16 pairs (lower k in the low half), round to nearest even
            float v[32];
            load_a_row<MODE>(A_hi(s), t128, v);
            uint32_t pk[16];
#pragma unroll
            for (int i = 0; i < 16; ++i) {
              __nv_bfloat162 pr = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
              pk[i] = *reinterpret_cast<uint32_t*>(&pr);
            }
            tmem_st16u(tmem_base + ((uint32_t)((warp & 3) * 32) << 16) + CF::kACol0 + st * CF::kAStride, pk);
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
          } else if (CF::kTmemA) {
            float v[32];
            load_a_row<MODE>(A_hi(s), t128, v);
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = tf32_rn(v[i]);
            tmem_st32(tmem_base + ((uint32_t)((warp & 3) * 32) << 16) + CF::kACol0 + st * CF::kAStride, v);
            asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
          }
        } else if (CF::kTmemA) {
          // thread t128 owns A row t128 = TMEM lane (quadrant warp % 4)
          float v[32], h[32];
          load_a_row<MODE>(A_hi(s), t128, v);
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            h[i] = tf32_rn(v[i]);
            v[i] = tf32_rn(v[i] - h[i]);
          }
          const uint32_t ta = tmem_base + ((uint32_t)((warp & 3) * 32) << 16) + CF::kACol0 + st * CF::kAStride;
          tmem_st32(ta, h);
          tmem_st32(ta + BK, v);
          asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
        } else {
          split_inplace((float4*)A_hi(s), (float4*)A_lo(s), CF::kABytes / 16, t128, 128);
        }
        if (MODE == 1 && !sh.one) split_inplace((float4*)B_hi(s), (float4*)B_lo(s), CF::kBBytes / 16, t128, 128);
        fence_proxy_async();
        tc_fence_before();
        if (PAIR == 2) {
          // this CTA's A half (TMEM / smem) and B half (landed: full[s]) are
          // ready: one release arrival per warp on the leader's barrier
          __syncwarp();
          if (lane == 0) mbar_arrive_cluster(conv_leader + (uint32_t)(cs * sizeof(uint64_t)));
        } else {
          mbar_arrive(&conv[cs]);
          if (threadIdx.x == 128) TCTRACE(2, kc);
        }
      }
    }
  } else if (warp >= 8) {
    const int q = warp & 3;                    // TMEM lane quadrant of this warp
    const int half = (warp - 8) >> 2;          // column half (chunks 32 apart)
    float* tb = epi_smem + (warp - 8) * 1280;   // 32 x 33 transpose tile / 32 x 32 TMA box
    const uint32_t tempty_leader = PAIR == 2 ? mapa_u32(smem_u32(tempty), 0) : 0u;
    int it = 0;
    for (int t = cta0; t < total; t += ncta, ++it) {
      int64_t kbeg;
      const int nkb = tile_kb(t, kbeg);
      const int z = t / tiles_mn, rem = t % tiles_mn;
      const int64_t m0 = (int64_t)(rem / sh.tiles_n) * (BM * PAIR) + (int64_t)rank * BM;
      const int64_t n0 = (int64_t)(rem % sh.tiles_n) * BN;
      const int acc = it & 1;
      mbar_wait_sleep(&tfull[acc], (it >> 1) & 1);
      if (threadIdx.x == 256) TCTRACE(5, it);
      tc_fence_after();
      float* Cz = C + (int64_t)z * sh.M * ldc;
      const int64_t row0 = m0 + q * 32;
#pragma unroll 1
      for (int c0 = 32 * half; c0 < BN; c0 += 32 * (EW / 4)) {
        if (n0 + c0 >= sh.N) break;
        uint32_t r[32];
        if (nkb > 0) {
          const uint32_t a0 = tmem_base + acc * (CF::kNAcc * CF::kAccCols) + ((uint32_t)(q * 32) << 16) +
                              (uint32_t)c0;
          tmem_ld32(a0, r);
#pragma unroll
          for (int pa = 1; pa < CF::kNAcc; ++pa) {   // fixed-order sum of the partial accumulators
            uint32_t r2[32];
            tmem_ld32(a0 + pa * CF::kAccCols, r2);
#pragma unroll
            for (int i = 0; i < 32; ++i) r[i] = __float_as_uint(__uint_as_float(r[i]) + __uint_as_float(r2[i]));
          }
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i) r[i] = 0;
        }
        // lane owns row (row0 + lane): epilogue in registers — the mask row
        // segment is read as 8 independent 128-bit loads per lane — then
        // either a TMA store of the 32 x 32 block or a transpose through smem
        // and column-coalesced stores.
        float v[32];
#pragma unroll
        for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
        if (MODE == 0 && epi.flags) {
          const int64_t row = row0 + lane;
          if (epi.flags & RDM_EPI_BIAS) {
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if (n0 + c0 + i < sh.N) v[i] += __ldg(epi.bias + n0 + c0 + i);
          }
          if (epi.flags & RDM_EPI_RELU) {
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = fmaxf(v[i], 0.f);
          }
          if ((epi.flags & RDM_EPI_MASK) && row < sh.M && epi.mask_bits) {
            const uint32_t mb = __ldg(epi.mask_bits + row * epi.ld_mask_bits + ((n0 + c0) >> 5));
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = (mb >> i) & 1u ? v[i] : 0.f;
          } else if ((epi.flags & RDM_EPI_MASK) && row < sh.M) {
            const float4* mrow = reinterpret_cast<const float4*>(epi.mask + row * epi.ld_mask + n0 + c0);
            float4 mk[8];
#pragma unroll
            for (int j = 0; j < 8; ++j)
              mk[j] = (n0 + c0 + 4 * j < sh.N) ? __ldg(mrow + j) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              v[4 * j + 0] = mk[j].x > 0.f ? v[4 * j + 0] : 0.f;
              v[4 * j + 1] = mk[j].y > 0.f ? v[4 * j + 1] : 0.f;
              v[4 * j + 2] = mk[j].z > 0.f ? v[4 * j + 2] : 0.f;
              v[4 * j + 3] = mk[j].w > 0.f ? v[4 * j + 3] : 0.f;
            }
          }
        }
        if (MODE == 0 && epi.bits_out && row0 + lane < sh.M) {
          uint32_t mb = 0;
#pragma unroll
          for (int i = 0; i < 32; ++i) mb |= (n0 + c0 + i < sh.N && v[i] > 0.f) ? (1u << i) : 0u;
          epi.bits_out[(row0 + lane) * epi.ld_bits_out + ((n0 + c0) >> 5)] = mb;
        }
        if (MODE == 0 && epi.twin) {
          const int64_t row = row0 + lane;
          if (row < sh.M) {
            const float sc = epi.twin_scale ? __ldg(epi.twin_scale + row) : 1.f;
            uint4* dst = reinterpret_cast<uint4*>(epi.twin + row * epi.ld_twin + n0 + c0);
            const int64_t cmax = epi.ld_twin - (n0 + c0);   // columns of this chunk inside the copy
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              if (8 * j >= cmax) break;
              uint32_t w[4];
#pragma unroll
              for (int h = 0; h < 4; ++h) {
                const int i = 8 * j + 2 * h;
                const float a = (n0 + c0 + i < sh.N) ? v[i] * sc : 0.f;
                const float b = (n0 + c0 + i + 1 < sh.N) ? v[i + 1] * sc : 0.f;
                __nv_bfloat162 pr = __floats2bfloat162_rn(a, b);
                w[h] = *reinterpret_cast<uint32_t*>(&pr);
              }
              dst[j] = make_uint4(w[0], w[1], w[2], w[3]);
            }
          }
        }
        if (sh.tstore) {
          // the lane's row as 8 float4 chunks of the 128-byte-swizzled box
          // (chunk j of row r at j ^ (r & 7): conflict-free); the TMA engine
          // writes the 32 x 32 block, clipping rows ≥ M and columns ≥ N
          if (lane == 0) bulk_wait_read0();   // the previous box has left shared memory
          __syncwarp();
          float4* box = reinterpret_cast<float4*>(tb);
#pragma unroll
          for (int j = 0; j < 8; ++j)
            box[lane * 8 + (j ^ (lane & 7))] = make_float4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]);
          fence_proxy_async();
          __syncwarp();
          if (lane == 0 && !(sh.dbg & 4)) {
            tma_store_2d(&tmC, tb, (int)(n0 + c0), (int)row0);
            bulk_commit();
          }
          continue;
        }
#pragma unroll
        for (int i = 0; i < 32; ++i) tb[lane * 33 + i] = v[i];
        __syncwarp();
        const int64_t col = n0 + c0 + lane;
        if (col < sh.N && !(sh.dbg & 4)) {
          const int nrows = (sh.M - row0) < 32 ? (int)(sh.M - row0) : 32;
#pragma unroll 8
          for (int rr = 0; rr < nrows; ++rr) Cz[(row0 + rr) * ldc + col] = tb[rr * 33 + lane];
          if (MODE == 0 && epi.scat.P) {
            // the same coalesced rows, stored into the owner of column `col`
            // (its column slice keeps global rows: my_off + row)
            const Scatter& s = epi.scat;
            int q = 0;
            while (q + 1 < s.P && s.lo[q + 1] <= col) ++q;
            const int64_t ldq = s.ld[q];
            float* d = s.ptr[q] + (s.my_off + row0) * ldq + (col - s.lo[q]);
#pragma unroll 8
            for (int rr = 0; rr < nrows; ++rr) d[rr * ldq] = tb[rr * 33 + lane];
          }
        }
        __syncwarp();
      }
      tc_fence_before();
      if (PAIR == 2) {
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(tempty_leader + (uint32_t)(acc * sizeof(uint64_t)));
      } else {
        mbar_arrive(&tempty[acc]);
        if (threadIdx.x == 256) TCTRACE(6, it);
      }
    }
    if (sh.tstore && lane == 0) bulk_wait0();   // every TMA store of this warp has landed
  }
  tc_fence_before();
  __syncthreads();
  if (PAIR == 2) {
    cluster_sync_all();   // the peer's MMAs (reading this CTA's smem / TMEM) are done
    if (warp == 2)
      asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base),
                   "n"(CF::kTmemCols));
  } else if (warp == 2) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base),
                 "n"(CF::kTmemCols));
  }
}

// B panels for NN / NT: Bt[n][kk] (K-major, row length ldb4) as hi and lo.
//  NN: B[kk][n] = W[kk][n]  → Bt[n][kk] = W[kk*ldw + n]   (W is K x N)
//  NT: B[kk][n] = W[n][kk]  → Bt[n][kk] = W[n*ldw + kk]   (W is N x K)
__global__ void prep_b_kernel(const float* __restrict__ W, int64_t ldw, int64_t K, int64_t N,
                              int transpose, float* __restrict__ hi, float* __restrict__ lo,
                              int64_t ldb) {
  const int64_t total = N * ldb;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = i / ldb, kk = i % ldb;
    float x = 0.f;
    if (kk < K) x = transpose ? W[kk * ldw + n] : W[n * ldw + kk];
    const float h = tf32_rn(x);
    hi[i] = h;
    lo[i] = tf32_rn(x - h);
  }
}

// bf16 B panels for the fast variant's kind::f16 GEMM: Bt[n][kk] (K-major, row
// length ldb, columns [K, ldb) zero), rounded to nearest even.
__global__ void prep_b_bf16_kernel(const float* __restrict__ W, int64_t ldw, int64_t K, int64_t N, int transpose,
                                   __nv_bfloat16* __restrict__ bt, int64_t ldb) {
  const int64_t total = N * ldb;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t n = i / ldb, kk = i % ldb;
    float x = 0.f;
    if (kk < K) x = transpose ? W[kk * ldw + n] : W[n * ldw + kk];
    bt[i] = __float2bfloat16_rn(x);
  }
}

__global__ void splitk_sum(const float* __restrict__ part, int splits, int64_t M, int64_t N,
                           int64_t ldp, float* __restrict__ C, int64_t ldc) {
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= M * N) return;
  const int64_t i = idx / N, n = idx % N;
  double s = 0.0;   // fixed order, fp64: the split partials of a long reduction
  const float* p = part + i * ldp + n;
  const int64_t zs = M * ldp;
  int z = 0;
  for (; z + 8 <= splits; z += 8) {   // 8 independent loads in flight, then the ordered adds
    float v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldcs(p + (int64_t)(z + u) * zs);
#pragma unroll
    for (int u = 0; u < 8; ++u) s += (double)v[u];
  }
  for (; z < splits; ++z) s += (double)__ldcs(p + (int64_t)z * zs);
  C[i * ldc + n] = (float)s;
}

// ------------------------------------------------------------ host side
PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    RDM_CUDA(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q));
    if (q != cudaDriverEntryPointSuccess || !p)
      throw Error(RDM_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
    fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
  }
  return fn;
}

// 2-D fp32 tensor map: inner dim (contiguous) x outer dim, row stride ld
// elements, box {box_inner, box_outer}, 128-byte swizzle, OOB → zeros.
CUtensorMap make_map(const float* base, int64_t inner, int64_t outer, int64_t ld, int box_inner,
                     int box_outer, CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  CUtensorMap m;
  cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)outer};
  cuuint64_t strides[1] = {(cuuint64_t)(ld * 4)};
  cuuint32_t box[2] = {(cuuint32_t)box_inner, (cuuint32_t)box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = encode_fn()(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void*)base, dims, strides, box,
                           es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS)
    throw Error(RDM_ERR_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
  return m;
}

template <int BN, int MODE, int EW, int PAIR, int ASM, int F16 = 0>
void launch_tc_ew(rdm_ctx* ctx, const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& blo,
               float* C, int64_t ldc, int64_t M, int64_t N, int64_t K, int splits, int n_mma,
               const TcEpi& e, const CUtensorMap* apf = nullptr) {
  using CF = Cfg<BN, EW, PAIR, ASM, F16>;
  auto kern = gemm_tc_kernel<BN, MODE, EW, PAIR, ASM, F16>;
  RDM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, CF::kSmem));
  TcShape sh;
  sh.M = M;
  sh.N = N;
  sh.K = K;
  sh.k_per_split = ceil_div(ceil_div(K, splits), BK) * BK;
  sh.tiles_m = (int)ceil_div(M, BM * PAIR);
  sh.tiles_n = (int)ceil_div(N, BN);
  sh.splits = splits;
  sh.n_mma = n_mma;
  sh.pf = apf != nullptr;
  const char* dbg = getenv("RDM_TC_DBG");
  sh.dbg = dbg ? atoi(dbg) : 0;
  sh.one = ctx->prec == RDM_PREC_FAST ? 1 : 0;
  // TMA-store epilogue: plain row-major output (one split, no fused scatter)
  // (TMA needs a 16-byte aligned base and a row pitch that is a multiple of
  // 16 bytes; other outputs take the transpose-and-store path)
  sh.tstore = (MODE == 0 && splits == 1 && !e.scat.P && ((uintptr_t)C & 15) == 0 && (ldc & 3) == 0 &&
               !(getenv("RDM_NO_TSTORE") && atoi(getenv("RDM_NO_TSTORE"))))
                  ? 1 : 0;
  const CUtensorMap tc = sh.tstore ? make_map(C, N, M, ldc, 32, 32) : a;
  const int64_t total = (int64_t)sh.tiles_m * sh.tiles_n * splits;
  if (PAIR == 1) {
    const unsigned grid = (unsigned)std::min<int64_t>(total, ctx->num_sms);
    kern<<<grid, CF::kThreads, CF::kSmem, ctx->stream>>>(a, b, blo, apf ? *apf : a, tc, C, ldc, sh, e);
  } else {
    // clusters of 2 CTAs (one CTA pair per TPC); the persistent grid is the
    // number of pairs that are co-resident (a GPC with an odd number of free
    // SMs leaves one idle: a grid of num_sms / 2 pairs would run a second wave)
    cudaLaunchConfig_t cfg{};
    cfg.blockDim = dim3(CF::kThreads);
    cfg.dynamicSmemBytes = CF::kSmem;
    cfg.stream = ctx->stream;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 2;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    static int max_pairs = 0;   // per instantiation
    if (max_pairs == 0) {
      cfg.gridDim = dim3((unsigned)ctx->num_sms);
      int n = 0;
      RDM_CUDA(cudaOccupancyMaxActiveClusters(&n, kern, &cfg));
      max_pairs = std::max(1, std::min(n, ctx->num_sms / 2));
      if (getenv("RDM_PAIR_LOG")) fprintf(stderr, "rdm: gemm pair BN=%d EW=%d: %d co-resident pairs\n", BN, EW, n);
    }
    cfg.gridDim = dim3((unsigned)(2 * std::min<int64_t>(total, max_pairs)));
    const CUtensorMap apm = apf ? *apf : a;
    RDM_CUDA(cudaLaunchKernelEx(&cfg, kern, a, b, blo, apm, tc, C, ldc, sh, e));
  }
  RDM_LAUNCHED(ctx);
}

// 2-D bf16 tensor map with the 64-byte swizzle (the fast GEMM's B panels: one
// 32-wide k-block is 64 bytes per row)
CUtensorMap make_map_bf16(const __nv_bfloat16* base, int64_t inner, int64_t outer, int64_t ld, int box_inner,
                          int box_outer) {
  CUtensorMap m;
  cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)outer};
  cuuint64_t strides[1] = {(cuuint64_t)(ld * 2)};
  cuuint32_t box[2] = {(cuuint32_t)box_inner, (cuuint32_t)box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = encode_fn()(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, (void*)base, dims, strides, box, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_64B,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS)
    throw Error(RDM_ERR_CUDA, "cuTensorMapEncodeTiled (bf16) failed (" + std::to_string((int)r) + ")");
  return m;
}

template <int BN, int MODE, int PAIR = 1, int ASM = 0>
void launch_tc(rdm_ctx* ctx, const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& blo,
               float* C, int64_t ldc, int64_t M, int64_t N, int64_t K, int splits, int n_mma,
               const TcEpi& e, const CUtensorMap* apf = nullptr) {
  // short contractions produce a wide output per k-block: epilogue-bound
  if (BN <= 128 && K <= 256)
    launch_tc_ew<BN, MODE, 8, PAIR, ASM>(ctx, a, b, blo, C, ldc, M, N, K, splits, n_mma, e, apf);
  else
    launch_tc_ew<BN, MODE, 4, PAIR, ASM>(ctx, a, b, blo, C, ldc, M, N, K, splits, n_mma, e, apf);
}

// CTA pairs for the row-sliced NN / NT products: every SM loads half of the W
// panel per row it computes (the 602-wide contractions are bound by each SM's
// ingress of A plus the re-read W panel).  Off for narrow outputs (BN < 32:
// the pair's N must be a multiple of 32) and for grids that would not fill the
// GPU's pairs.  RDM_PAIR=0 / 1 forces either (experiments).
// Measured per call (tools/time_gemm.py, profiles/r2_gemm_pair.md): BN = 256
// pairs (A in smem) 1.61 → 1.32 ms for the products-shaped 2.45 M x 256 · 256
// x 256; BN ≤ 128 with A in TMEM gains where K is short and N ≤ 256 (K = 100,
// N = 256: 1.10 → 1.02 ms), with A split in smem and two partial accumulators
// where K is long or the tile narrow (K = 602: 229 → 208 µs; N = 41: 68 → 52
// µs); the 602-wide NT (K = 128, five 128-wide tiles) and single-tile short
// contractions stay single.
// Returns 0 (single CTA), 1 (pair, A in TMEM / smem for BN = 256), 2 (pair, A
// split in smem, BN ≤ 128); pairs only from 148·256 rows on.
int use_pair(rdm_ctx* ctx, int64_t M, int64_t N, int64_t K, int BN, int splits) {
  if (BN < 32 || splits > 1) return 0;
  const char* fp = getenv("RDM_PAIR");
  const char* fa = getenv("RDM_PAIR_ASMEM");
  if (fp && !atoi(fp)) return 0;
  // at least two 256-row pair tiles per SM pair: the GraphSAINT subgraphs
  // (≈ 25 k rows, GEMMs running beside the sampler's kernels on its own
  // stream) ran 3.74 → 3.85 ms per step with pairs, which need whole TPCs free
  if (!fp && M < (int64_t)ctx->num_sms * 2 * BM) return 0;
  if (BN == 256) return 1;
  if (fa) return atoi(fa) ? 2 : 1;
  if (K >= 256 || BN <= 64) return 2;
  // two 128-wide tiles (products-shaped 100 → 256): A in TMEM; one tile of a
  // short contraction (the Reddit-shaped NT 41 → 128 with its mask: 75 vs 82
  // µs in the epoch's launch list) and the five tiles of the 602-wide NT stay single
  if ((N > BN && N <= 256) || fp) return 1;
  return 0;
}

// Wider N: one 256-wide tile (A in smem, both TMEM accumulators) where the
// contraction is long enough for the 3xTF32 MMAs to dominate (measured,
// tools/time_gemm.py, products-shaped 2.45 M x 256 · 256 x 256: 1.94 →
// 1.76 ms), else several 128-wide tiles (TMEM-A path; K = 100: 1.18 vs
// 1.47 ms).  RDM_BN256=1 / 0 forces either (experiments).
int pick_bn(int64_t N, int64_t K = 0, bool three = true, bool mask = false, bool pairs = false) {
  if (N <= 16) return 16;
  if (N <= 32) return 32;
  if (N <= 64) return 64;
  if (N <= 128) return 128;
  if (const char* e = getenv("RDM_BN256")) return atoi(e) ? 256 : 128;
  // (a Hadamard-mask epilogue over 256 columns with 4 epilogue warps loses
  // more than the wide tile gains: 1.06 → 1.34 ms in the products epoch)
  if (!three) return 128;
  // 256-wide tiles on CTA pairs pay at short K and with the Hadamard mask too
  // (profiles/r2_gemm_pair.md: the Reddit-shaped 602-wide NT, K = 128, 243 →
  // 205 µs; products-shaped NN 100 → 256 1.12 → 0.83 ms; the products epoch
  // with its masked NT 256 → 256 on 256-wide pair tiles 41.44 → 40.82 ms);
  // single CTAs only from K = 256 on and without a mask
  if (pairs) return 256;
  return (K >= 256 && !mask) ? 256 : 128;
}

}  // namespace

namespace {
// Fast variant, NN / NT: bf16 operands on kind::f16 (twice the tf32 MMA rate,
// half the W panel bytes); A stays fp32 in HBM and is rounded by the converter.
// RDM_F16_GEMM=0 keeps the 1xTF32 kernel (experiments).
bool use_f16_gemm(rdm_ctx* ctx) {
  if (ctx->prec != RDM_PREC_FAST) return false;
  const char* e = getenv("RDM_F16_GEMM");
  return !e || atoi(e) != 0;
}

void launch_nn_bf16(rdm_ctx* ctx, const float* X, int64_t ldx, const __nv_bfloat16* bt, int64_t ldb, float* C,
                    int64_t ldc, int64_t M, int64_t N, int64_t K, const TcEpi& e) {
  const int BN = pick_bn(N, 0, false);
  const int nm = N > BN ? BN : (int)(((N + 15) / 16) * 16);
  const CUtensorMap ta = make_map(X, K, M, ldx, BK, BM);
  const CUtensorMap tb = make_map_bf16(bt, K, N, ldb, BK, BN);
  switch (BN) {
#define RDM_F16_CASE(B)                                                                        \
  case B:                                                                                      \
    if (K <= 256) launch_tc_ew<B, 0, 8, 1, 0, 1>(ctx, ta, tb, tb, C, ldc, M, N, K, 1, nm, e); \
    else launch_tc_ew<B, 0, 4, 1, 0, 1>(ctx, ta, tb, tb, C, ldc, M, N, K, 1, nm, e);          \
    break;
    RDM_F16_CASE(16)
    RDM_F16_CASE(32)
    RDM_F16_CASE(64)
    default: RDM_F16_CASE(128)
#undef RDM_F16_CASE
  }
}

void launch_nn_panels(rdm_ctx* ctx, const float* X, int64_t ldx, const float* bhi, const float* blo,
                      int64_t ldb, float* C, int64_t ldc, int64_t M, int64_t N, int64_t K,
                      const TcEpi& e, int splits = 1, bool wide_ok = true) {
  // (256-wide tiles only for single-split calls: the split-K hub-core GEMM of
  // the GraphSAINT subgraphs ran slower with them)
  // would a 256-wide tile run on CTA pairs (use_pair's row threshold)?
  const bool pairs_ok = splits == 1 && use_pair(ctx, M, N, K, 256, 1) != 0;
  const int BN = (splits == 1 && wide_ok) ? pick_bn(N, K, ctx->prec != RDM_PREC_FAST, (e.flags & RDM_EPI_MASK) != 0,
                                                    pairs_ok)
                                         : pick_bn(N, 0, false);
  const int pmode = use_pair(ctx, M, N, K, BN, splits);
  const bool pair = pmode != 0;
  // one MMA width for every tile: BN when N spans several tiles, else N rounded
  // to 16 (to 32 for a pair, whose CTAs load nm/2 rows of B each)
  const int nm = N > BN ? BN : pair ? (int)(((N + 31) / 32) * 32) : (int)(((N + 15) / 16) * 16);
  const CUtensorMap ta = make_map(X, K, M, ldx, BK, BM);
  const CUtensorMap tb = make_map(bhi, K, N, ldb, BK, pair ? nm / 2 : BN);
  const CUtensorMap tbl = make_map(blo, K, N, ldb, BK, pair ? nm / 2 : BN);
  // L2-prefetch map: 128 x 128 fp32 boxes (512-byte row segments), no swizzle
  // (off by default: measured at the end of round 1, tools/time_gemm.py, the
  // 232,965 x 602 · 602 x 128 NN runs 231 → 225 µs fp32 and 175 → 150 µs fast
  // without it; RDM_PF=1 re-enables it for experiments)
  const bool pf = K > 4 * BK && getenv("RDM_PF") && atoi(getenv("RDM_PF"));
  const CUtensorMap tpf = pf ? make_map(X, K, M, ldx, 4 * BK, BM, CU_TENSOR_MAP_SWIZZLE_NONE) : ta;
  const CUtensorMap* p = pf ? &tpf : nullptr;
  if (pmode == 2) {
    switch (BN) {
      case 64: launch_tc<64, 0, 2, 1>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); return;
      case 128: launch_tc<128, 0, 2, 1>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); return;
      default: break;
    }
  }
  if (pair) {
    switch (BN) {
      case 32: launch_tc<32, 0, 2>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
      case 64: launch_tc<64, 0, 2>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
      case 128: launch_tc<128, 0, 2>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
      default: launch_tc<256, 0, 2>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
    }
    return;
  }
  switch (BN) {
    case 16: launch_tc<16, 0>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
    case 32: launch_tc<32, 0>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
    case 64: launch_tc<64, 0>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
    case 128: launch_tc<128, 0>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
    default: launch_tc<256, 0>(ctx, ta, tb, tbl, C, ldc, M, N, K, splits, nm, e, p); break;
  }
}
}  // namespace

void gemm_tc_panels(rdm_ctx* ctx, const float* A, int64_t lda, const float* bhi, const float* blo,
                    int64_t ldb, float* C, int64_t ldc, int64_t M, int64_t N, int64_t K) {
  RDM_CHECK_ARG(!((uintptr_t)A & 15) && !(lda & 3) && !((uintptr_t)bhi & 15) &&
                    !((uintptr_t)blo & 15) && !(ldb & 3),
                "gemm_tc_panels: 16-byte aligned operands with ld % 4 == 0 required");
  // Split K so that the persistent grid has no idle SMs (the hub-core GEMM has
  // only ~110 M-tiles for 148 SMs); partial slabs are summed in split order.
  const int64_t tiles = ceil_div(M, BM) * ceil_div(N, pick_bn(N, 0, false));
  int best_s = 1;
  double best_eff = 0;
  for (int s = 1; s <= 8; ++s) {
    if (s > 1 && K / s < 16 * BK) break;
    const int64_t t = tiles * s;
    const double eff = (double)t / (double)(ctx->num_sms * ceil_div(t, ctx->num_sms));
    if (eff > best_eff + 0.02) {
      best_eff = eff;
      best_s = s;
    }
  }
  if (best_s == 1) {
    launch_nn_panels(ctx, A, lda, bhi, blo, ldb, C, ldc, M, N, K, TcEpi{0, nullptr, nullptr, 0}, 1, false);
    return;
  }
  const int64_t ldo = roundup4(N);
  float* part = ensure_ws(ctx->ws_gemm, (size_t)best_s * M * ldo * sizeof(float));
  launch_nn_panels(ctx, A, lda, bhi, blo, ldb, part, ldo, M, N, K, TcEpi{0, nullptr, nullptr, 0}, best_s);
  splitk_sum<<<(unsigned)ceil_div(M * N, 256), 256, 0, ctx->stream>>>(part, best_s, M, N, ldo, C, ldc);
  RDM_LAUNCHED(ctx);
}

static bool g_tc_disabled = false;

bool gemm_tc(rdm_ctx* ctx, int op, const float* X, int64_t ldx, const float* W, int64_t ldw,
             float* C, int64_t ldc, int64_t rows, int64_t k, int64_t m, int epi, const float* bias,
             const float* mask, const Scatter* scat) {
  if (g_tc_disabled) return false;
  // TMA: global base 16-byte aligned, row strides multiples of 16 bytes
  if (((uintptr_t)X & 15) || (ldx & 3)) return false;
  // the epilogue reads mask rows as float4: 16-byte aligned rows required
  if ((epi & RDM_EPI_MASK) && (((uintptr_t)mask & 15) || (ldc & 3))) return false;
  TcEpi e{epi, bias, mask, ldc, Scatter{}};
  if (op == RDM_GEMM_NN || op == RDM_GEMM_NT) {
    if (scat) e.scat = *scat;
    e.bits_out = ctx->gemm_bits_out;
    e.ld_bits_out = ctx->gemm_bits_ld;
    e.mask_bits = ctx->gemm_mask_bits;
    e.ld_mask_bits = ctx->gemm_mask_bits_ld;
    if (ctx->gemm_bits_out) ctx->gemm_bits_written = true;
    if (ctx->gemm_twin) {
      e.twin = static_cast<uint16_t*>(ctx->gemm_twin);
      e.ld_twin = ctx->gemm_twin_ld;
      e.twin_scale = ctx->gemm_twin_scale;
      ctx->gemm_twin_written = true;
    }
    const int64_t M = rows;
    const int64_t N = op == RDM_GEMM_NN ? m : k;   // output columns
    const int64_t K = op == RDM_GEMM_NN ? k : m;   // contraction
    if (use_f16_gemm(ctx)) {
      // rows padded to 128 bytes (zeros past K): an unaligned panel pitch (K = 100:
      // 208 B) made every 64-byte box row straddle sectors — 0.69 → 1.0 ms
      const int64_t ldb16 = (K + 63) / 64 * 64;
      __nv_bfloat16* bt =
          reinterpret_cast<__nv_bfloat16*>(ensure_ws(ctx->ws_tcb, (size_t)N * ldb16 * sizeof(__nv_bfloat16)));
      prep_b_bf16_kernel<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(N * ldb16, 256), 4096)), 256,
                           0, ctx->stream>>>(W, ldw, K, N, op == RDM_GEMM_NN ? 1 : 0, bt, ldb16);
      RDM_LAUNCHED(ctx);
      launch_nn_bf16(ctx, X, ldx, bt, ldb16, C, ldc, M, N, K, e);
      return true;
    }
    // (128-byte panel rows, as the bf16 path uses, measured within noise here)
    const int64_t ldb = roundup4(K);
    float* bws = ensure_ws(ctx->ws_tcb, (size_t)2 * N * ldb * sizeof(float));
    float* bhi = bws;
    float* blo = bws + N * ldb;
    prep_b_kernel<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(N * ldb, 256), 4096)), 256, 0,
                    ctx->stream>>>(W, ldw, K, N, op == RDM_GEMM_NN ? 1 : 0, bhi, blo, ldb);
    RDM_LAUNCHED(ctx);
    launch_nn_panels(ctx, X, ldx, bhi, blo, ldb, C, ldc, M, N, K, e);
    return true;
  }
  // TN: C[k x m] = Xᵀ U  (X rows x k at ldx, U rows x m at ldw)
  if (scat) return false;   // weight gradients are never redistributed
  if (((uintptr_t)W & 15) || (ldw & 3)) return false;
  const int64_t M = k, N = m, K = rows;
  // TN: 256-wide tiles for N > 128 (products-shaped 256 x 256 over 2.45 M rows:
  // 1.89 → 1.71 ms fp32, 0.96 → 0.92 ms fast)
  const int BN = N <= 32 ? 32 : N <= 64 ? 64 : N <= 128 ? 128
                 : (getenv("RDM_BN256") ? (atoi(getenv("RDM_BN256")) ? 256 : 128) : 256);
  const int n_mma = (int)std::min<int64_t>(BN, ((N + 31) / 32) * 32);
  // CTA pairs (M = 256 per pair, each CTA loading half of U's 32-wide chunks):
  // every SM loads half the U bytes per row chunk and the MMAs read half of B
  // from its smem.  Needs M ≥ 256 and halves of whole 32-wide chunks.
  const char* tp = getenv("RDM_TN_PAIR");
  // Only where the 256-row pair tiles cover M with little padding: products-
  // shaped 256 x 256 1.91 → 1.29 ms, while the 602-wide Reddit-shaped one (a
  // third pair tile of 90 rows) went 236 → 276 µs (profiles/r2_gemm_pair.md).
  const bool tile_fit = ceil_div(M, 2 * BM) * 2 * BM - M <= M / 10;
  const bool pair = !(tp && !atoi(tp)) && M >= 2 * BM && BN >= 64 && n_mma % 64 == 0 &&
                    ((K >= (int64_t)ctx->num_sms * 2 * BM && tile_fit) || (tp && atoi(tp)));   // RDM_TN_PAIR=1: forced (tests)
  const int64_t tiles = ceil_div(M, BM * (pair ? 2 : 1)) * ceil_div(N, BN);
  const int64_t slots = pair ? ctx->num_sms / 2 : ctx->num_sms;
  int64_t splits = std::max<int64_t>(1, slots / std::max<int64_t>(1, tiles));
  // accuracy: the weight gradient sums over every row, often with heavy
  // cancellation (softmax − onehot is zero-sum); chains of at most kTnChain
  // rows in the fp32 TMEM accumulator (kTnChain), the partials summed in fp64
  // (splitk_sum): products-shaped Y^3 over 2.45 M rows 1.6e-4 → within 1e-4
  int64_t chain = 4096;
  if (const char* e = getenv("RDM_TN_CHAIN")) chain = std::max<int64_t>(256, atoll(e));
  splits = std::max<int64_t>(splits, ceil_div(K, chain));
  // as many splits as the rounds of the persistent grid hold anyway (shorter
  // chains, no idle slots in the last round)
  splits = std::max<int64_t>(splits, ceil_div(tiles * splits, slots) * slots / tiles);
  splits = std::min<int64_t>(splits, std::max<int64_t>(1, K / (8 * BK)));
  const CUtensorMap ta = make_map(X, M, K, ldx, 32, BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B);  // inner = k
  const CUtensorMap tb = make_map(W, N, K, ldw, 32, BK, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B);  // inner = m
  float* out = C;
  int64_t ldo = ldc;
  if (splits > 1) {
    ldo = roundup4(N);
    out = ensure_ws(ctx->ws_gemm, (size_t)splits * M * ldo * sizeof(float));
  }
  TcEpi none{0, nullptr, nullptr, 0};
  if (pair) {
    const CUtensorMap tbh = tb;   // the same 32 x 32 chunk boxes; each CTA loads its half of the chunks
    switch (BN) {
      case 64: launch_tc<64, 1, 2>(ctx, ta, tbh, tbh, out, ldo, M, N, K, (int)splits, n_mma, none); break;
      case 128: launch_tc<128, 1, 2>(ctx, ta, tbh, tbh, out, ldo, M, N, K, (int)splits, n_mma, none); break;
      default: launch_tc<256, 1, 2>(ctx, ta, tbh, tbh, out, ldo, M, N, K, (int)splits, n_mma, none); break;
    }
  } else switch (BN) {
    case 32: launch_tc<32, 1>(ctx, ta, tb, tb, out, ldo, M, N, K, (int)splits, n_mma, none); break;
    case 64: launch_tc<64, 1>(ctx, ta, tb, tb, out, ldo, M, N, K, (int)splits, n_mma, none); break;
    case 128: launch_tc<128, 1>(ctx, ta, tb, tb, out, ldo, M, N, K, (int)splits, n_mma, none); break;
    default: launch_tc<256, 1>(ctx, ta, tb, tb, out, ldo, M, N, K, (int)splits, n_mma, none); break;
  }
  if (splits > 1) {
    splitk_sum<<<(unsigned)ceil_div(M * N, 256), 256, 0, ctx->stream>>>(out, (int)splits, M, N, ldo, C,
                                                                          ldc);
    RDM_LAUNCHED(ctx);
  }
  return true;
}

}  // namespace rdm

extern "C" int rdm_debug_tc_trace(long long* out, int n) {
#ifdef RDM_TC_TRACE
  const int m = n < 8 * rdm::kTrN ? n : 8 * rdm::kTrN;
  return cudaMemcpyFromSymbol(out, rdm::g_tc_trace, (size_t)m * sizeof(long long)) == cudaSuccess ? m : -1;
#else
  (void)out;
  (void)n;
  return 0;
#endif
}

extern "C" int rdm_debug_disable_tc(int disable) {
  rdm::g_tc_disabled = disable != 0;
  return 0;
}
