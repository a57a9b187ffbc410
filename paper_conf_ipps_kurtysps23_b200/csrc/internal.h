// internal.h — shared declarations of the rdm library (not part of the ABI).
#pragma once

#include <cuda_runtime.h>
#include <nccl.h>

#include <cstdint>
#include <map>
#include <memory>
#include <stdexcept>
#include <string>
#include <vector>

#include "../../include/rdm.h"

namespace rdm {

// ------------------------------------------------------------------ errors
struct Error : std::runtime_error {
  rdm_status status;
  Error(rdm_status s, const std::string& m) : std::runtime_error(m), status(s) {}
};

#define RDM_CHECK_ARG(cond, msg)                                      \
  do {                                                                \
    if (!(cond)) throw ::rdm::Error(RDM_ERR_ARG, std::string(msg));   \
  } while (0)

#define RDM_CUDA(call)                                                                     \
  do {                                                                                     \
    cudaError_t e_ = (call);                                                               \
    if (e_ != cudaSuccess)                                                                 \
      throw ::rdm::Error(e_ == cudaErrorMemoryAllocation ? RDM_ERR_OOM : RDM_ERR_CUDA,     \
                         std::string(#call) + ": " + cudaGetErrorString(e_) + " @" +       \
                             __FILE__ + ":" + std::to_string(__LINE__));                   \
  } while (0)

#define RDM_LAUNCHED(ctx)                                                                  \
  do {                                                                                     \
    cudaError_t e_ = cudaGetLastError();                                                   \
    if (e_ != cudaSuccess)                                                                 \
      throw ::rdm::Error(RDM_ERR_CUDA, std::string("kernel launch: ") +                    \
                                           cudaGetErrorString(e_) + " @" + __FILE__ + ":" + \
                                           std::to_string(__LINE__));                      \
    (ctx)->counters.kernel_launches++;                                                     \
    (ctx)->phase_launches[(ctx)->cur_phase]++;                                             \
  } while (0)

inline int64_t roundup4(int64_t x) { return (x + 3) & ~int64_t(3); }
inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// --------------------------------------------------------------- partition
struct Range {
  int64_t lo, hi;
  int64_t size() const { return hi - lo; }
};
Range row_range(int64_t n, int P, int p);
Range col_range(int64_t f, int P, int p);

// ------------------------------------------------------------ device memory
struct DevBuf {
  void* ptr = nullptr;
  size_t bytes = 0;
  DevBuf() = default;
  explicit DevBuf(size_t b);
  ~DevBuf();
  DevBuf(const DevBuf&) = delete;
  DevBuf& operator=(const DevBuf&) = delete;
  template <class T>
  T* as() const { return static_cast<T*>(ptr); }
};

// Buffers retired by a regrowth (ensure_ws / Pinned) inside a step: freeing
// them at once would synchronise the whole device, so they are parked here
// and released at the next host synchronisation point (rdm_sync, finalize,
// sampler / executor destruction).
void retire(void* dev_ptr, void* host_ptr);
void release_retired();

// Pinned host staging buffer (grows, never shrinks): D2H copies into pageable
// memory block the host at the call, and H2D copies from pageable memory are
// synchronous, so copies meant to stay asynchronous go through one of these.
// A regrowth retires the old buffer (freed at the next rdm_sync / finalize:
// cudaFreeHost synchronises the device) and is logged under RDM_WS_LOG.
struct Pinned {
  void* p = nullptr;
  size_t bytes = 0;
  Pinned() = default;
  Pinned(const Pinned&) = delete;
  Pinned& operator=(const Pinned&) = delete;
  Pinned(Pinned&& o) noexcept : p(o.p), bytes(o.bytes) {
    o.p = nullptr;
    o.bytes = 0;
  }
  Pinned& operator=(Pinned&& o) noexcept {
    if (this != &o) {
      if (p) retire(nullptr, p);
      p = o.p;
      bytes = o.bytes;
      o.p = nullptr;
      o.bytes = 0;
    }
    return *this;
  }
  ~Pinned();
  void reserve(size_t want);
  template <class T> T* get(size_t count) {
    reserve(count * sizeof(T));
    return static_cast<T*>(p);
  }
};

// ------------------------------------------------------------------- graph
struct Csr;

// Dense "hub core" of a symmetric adjacency: the K highest-degree vertices'
// mutual block A[hubs, hubs], stored dense (K x K fp32, hub slots in degree
// order) and multiplied on the tensor cores; the CSR `resid` holds every other
// entry.  A·X = resid·X + scatter_hub_rows(Acore · X[hubs]).
struct Core {
  int64_t K = 0;                       // hub count (multiple of 128), 0 = no core
  int64_t nnz = 0;                     // entries moved into the dense block
  bool forced = false;                 // RDM_CORE_K override: use at every width
  std::unique_ptr<DevBuf> A;           // K x K fp32, row-major
  std::unique_ptr<DevBuf> hub_ids;     // int32[K]: vertex of slot k
  std::unique_ptr<DevBuf> hub_slot;    // int32[N]: slot of vertex v, -1 if not a hub
  std::unique_ptr<Csr> resid;          // A minus the core entries (with its own bins)
  // Binary hub tiles (hubtiles.cu) — used instead of the dense block (K = 0)
  // when every value of the hub region factors as a_ij = s_i·s_j (the GCN
  // symmetric normalisation D^-1/2 (A+I) D^-1/2, or all ones): the region of
  // the K2 highest-degree vertices is cut into 128 x 128 rank blocks, blocks
  // dense enough to pay are stored as 0/1 bf16 tiles and multiplied on the
  // kind::f16 tensor cores against s_j·X_j split into three bf16 pieces.
  int64_t K2 = 0;                      // rank range covered (multiple of 128), 0 = none
  int64_t n_tiles = 0, n_items = 0, n_rb = 0;
  std::unique_ptr<DevBuf> tiles;       // bf16 [n_tiles][128][128], 0/1 (row = rank in block)
  std::unique_ptr<DevBuf> tile_cb;     // int32[n_tiles]: column block of each tile
  std::unique_ptr<DevBuf> item_tb;     // int32[n_items+1]: tile range of each work item
  std::unique_ptr<DevBuf> rb_item;     // int32[n_rb+1]: item range of each row block
  std::unique_ptr<DevBuf> scale;       // fp32[K2]: column scale c of the vertex of slot k (a_ij = r_i c_j)
  std::unique_ptr<DevBuf> rscale;      // fp32[K2]: row scale r of the vertex of slot k
  // pair items (int8 kernel): row blocks 2p, 2p+1 merged by column block
  int64_t n_pairs = 0, n_pitems = 0;
  std::unique_ptr<DevBuf> pm_cb, pm_t1, pm_t2;   // int32[merged]: column block, tile of 2p / 2p+1 (-1 none)
  std::unique_ptr<DevBuf> pitem_pm;              // int32[n_pitems+1]: merged range of each item
  std::unique_ptr<DevBuf> pair_item;             // int32[n_pairs+1]: item range of each pair
  std::unique_ptr<DevBuf> zero_bits;             // one all-zero tile (2 KB)
};

struct Csr {
  int64_t n = 0, nnz = 0;
  int64_t n_in = -1;   // rows of the dense input (columns of A); -1 = n (square)
  int64_t in_rows() const { return n_in < 0 ? n : n_in; }
  std::unique_ptr<DevBuf> rowptr, col, val;
  Core core;
  // row bins (see spmm.cu): light rows processed warp-per-row, heavy rows
  // split into fixed-size nnz segments reduced deterministically.
  int64_t n_light = 0, n_seg = 0, n_heavy = 0;
  // light rows by degree (light_rows is sorted by descending degree):
  // deg_ge[d] = number of light rows of degree >= d, d = 0..kDegTab (host copy)
  static constexpr int kDegTab = 128;
  int64_t deg_ge[kDegTab + 1] = {};
  std::unique_ptr<DevBuf> light_rows;   // int32[n_light], longest rows first
  std::unique_ptr<DevBuf> seg_start;    // int64[n_seg]: first nnz of each segment
  std::unique_ptr<DevBuf> heavy_rows;   // int32[n_heavy]
  std::unique_ptr<DevBuf> heavy_seg;    // int32[n_heavy+1]: segment range of heavy row
  Pinned bins_stage;                    // pinned staging of the bins' upload (build_bins)
  // column relabelling (spmm.cu build_hot): col_hot[j] = rank of col[j] by
  // reference count, hot_ids[rank] = vertex (hot_max = number of columns)
  int64_t hot_max = 0;
  std::unique_ptr<DevBuf> col_hot, hot_ids;
  int64_t max_deg = 0;
  // every stored value factors as a_ij = s_i·s_j (GCN normalisation; checked
  // on the host at rdm_set_graph): fp32 s per row, used by the fast-precision
  // SpMM (sum of bf16(s_j X_j), s_i in the epilogue); null otherwise
  std::unique_ptr<DevBuf> fscale;
};

struct Graph {
  int64_t n = 0, nnz = 0;
  bool symmetric = true;
  Csr A;    // rows of A: used for A·X (eq. 3-4)
  Csr AT;   // rows of Aᵀ: used for Aᵀ·X (eq. 1); empty if symmetric
  const Csr& fwd() const { return symmetric ? A : AT; }
  const Csr& bwd() const { return A; }
};

}  // namespace rdm

// --------------------------------------------------------------- context
struct rdm_ctx {
  int world = 1;
  int rank = 0;                  // RDM_ALL_RANKS for a virtual group
  std::vector<int> local;        // global ranks held in this process
  int device = 0;
  int num_sms = 148;
  cudaStream_t stream = nullptr;
  ncclComm_t comm = nullptr;
  bool poisoned = false;
  bool emulated = false;         // one rank of a P-rank job with no peers (rdm_init_emulated)
  int transport = 0;             // RDM_TRANSPORT_NCCL / RDM_TRANSPORT_P2P
  int prec = 0;                  // RDM_PREC_FP32 / RDM_PREC_FAST
  bool spmm_in_bf16 = false;     // executor → spmm: the input holds bf16 values (bf16 wire)
  // fast variant, cast folded into the producing GEMM (executor → gemm_tc):
  // the GEMM also writes a bf16 copy (row length gemm_twin_ld, rows × scale)
  void* gemm_twin = nullptr;
  int64_t gemm_twin_ld = 0;
  const float* gemm_twin_scale = nullptr;
  bool gemm_twin_written = false;
  // … and the SpMM that reads `bf16_twin_src` takes the copy instead of casting
  const float* bf16_twin_src = nullptr;
  bool bf16_twin_fact = false;
  // ReLU sign bits (executor → gemm_tc, NN/NT): write them for the output /
  // read the Hadamard from them; gemm_bits_written reports that the tensor-core
  // path (not the SIMT fallback) ran
  uint32_t* gemm_bits_out = nullptr;
  int64_t gemm_bits_ld = 0;
  const uint32_t* gemm_mask_bits = nullptr;
  int64_t gemm_mask_bits_ld = 0;
  bool gemm_bits_written = false;
  std::string err;
  rdm::Graph graph;
  bool has_graph = false;
  rdm_counters counters{};
  // workspace (grown on demand, never shrunk)
  std::vector<std::unique_ptr<rdm::DevBuf>> ws_send, ws_recv;  // per local slot
  std::unique_ptr<rdm::DevBuf> ws_seg;                         // SpMM heavy-row partials
  std::unique_ptr<rdm::DevBuf> ws_gemm;                        // GEMM split-K partials
  std::unique_ptr<rdm::DevBuf> ws_tcb;                         // tcgen05 B panels (hi | lo)
  std::unique_ptr<rdm::DevBuf> ws_stage;                       // host-input staging
  std::unique_ptr<rdm::DevBuf> ws_core_b, ws_core_c;           // hub-core panels / product
  std::unique_ptr<rdm::DevBuf> ws_scratch;
  // R_A < P (§III-E): row panels of A held by this process (index = panel id;
  // an NCCL rank holds its own panel only), the panel-group size R_A
  int panel_RA = 0;
  int64_t panel_n = 0;
  std::vector<std::unique_ptr<rdm::Csr>> panels;
  std::unique_ptr<rdm::DevBuf> ws_panel_in;                    // all-gathered N x w_j input per slot
  std::unique_ptr<rdm::DevBuf> ws_tile_cs;                     // fp16 hub tiles: column scales + maxima
  std::unique_ptr<rdm::DevBuf> ws_bf16;                        // RDM_PREC_FAST: bf16 copy of the SpMM input
  std::unique_ptr<rdm::DevBuf> ws_hot;                         // hot-row panel of the SpMM input
  // phase timing
  bool timing = false;
  int cur_phase = RDM_PH_OTHER;
  struct Ev {
    int phase;
    cudaEvent_t a, b;
  };
  std::vector<Ev> events;
  std::vector<cudaEvent_t> event_pool;
  // auxiliary stream: the SpMM's short-row kernel runs on it beside the
  // long-row kernel (disjoint rows), forked / joined with these events
  cudaStream_t aux = nullptr;
  cudaEvent_t aux_fork = nullptr, aux_join = nullptr;
  double phase_ms[RDM_PH_COUNT] = {};
  int64_t phase_launches[RDM_PH_COUNT] = {};
  bool virtual_group() const { return rank == RDM_ALL_RANKS && world > 1; }
  int nlocal() const { return (int)local.size(); }
};

// GraphSAINT-RDM sampler (saint.cu): the current subgraph and the device
// workspace that builds it.
struct rdm_saint {
  rdm_ctx* ctx = nullptr;
  rdm::Pinned h_scal, h_rp, h_rrp, h_bucket;   // host staging of the sampler's round trips
  bool reserved = false;  // every workspace sized at its bound (first rdm_saint_sample)
  int64_t roots = 0;
  int walk_len = 0;
  uint64_t seed = 0;
  int64_t n_cap = 0;
  int64_t nnz_bound = 0;  // entries of any subgraph (reserve_bounds)
  // Double-buffered subgraphs: rdm_saint_sample builds the next subgraph on the
  // sampler's own stream into the buffer the previous-but-one subgraph used
  // (after the executor released it, ev_free), while the compute stream still
  // trains on the current one; the executor waits for ev_done of the buffer it
  // switches to.
  rdm::Graph bufs[2];     // subgraphs (symmetric: A only)
  std::unique_ptr<rdm::DevBuf> nodes_b[2];   // sorted node list of each buffer
  int cur = 0;            // buffer of the latest sample
  cudaStream_t sst = nullptr;
  cudaEvent_t ev_done[2] = {nullptr, nullptr}, ev_free[2] = {nullptr, nullptr};
  bool freed[2] = {false, false};
  rdm::Graph& graph() { return bufs[cur]; }
  const rdm::Graph& graph() const { return bufs[cur]; }
  int64_t version = 0;    // bumped by every rdm_saint_sample
  int64_t iteration = -1;
  std::unique_ptr<rdm::DevBuf> visits, flag, map, deg, seg, rps, scal, tmp, mask_s;
  std::unique_ptr<rdm::DevBuf> core_tmp, core_rank, core_seg, core_cnt, core_bucket, tmp2;
};

namespace rdm {

float* ensure_ws(std::unique_ptr<DevBuf>& b, size_t bytes);

// Scoped phase timer: records CUDA events on the ctx stream around a phase.
struct Phase {
  rdm_ctx* ctx;
  int prev;
  cudaEvent_t a = nullptr;
  Phase(rdm_ctx* c, int ph);
  ~Phase();
};

// Fused redistribution ("p2p" transport): the producing kernel of a tensor
// that is redistributed next also stores every element straight into its
// owner's destination layout (peer memory over NVLink for NCCL ranks, the
// other slots' buffers in a virtual group), replacing pack + all-to-all.
struct Scatter {
  static constexpr int kMax = 64;
  int P = 0;                 // 0 = no scatter
  int mode = 0;              // 1: row slice → column slices (GEMM), 2: column slice → row slices (SpMM)
  int64_t lo[kMax + 1] = {}; // destination partition: columns (mode 1) / rows (mode 2)
  int64_t ld[kMax] = {};     // destination leading dim per rank
  float* ptr[kMax] = {};     // destination base per rank
  int64_t my_off = 0;        // mode 1: my first global row; mode 2: my first global column
  int64_t my_w = 0;          // mode 2: real width of my column slice
};

// ------------------------------------------------------------------ kernels
// spmm.cu
void spmm(rdm_ctx* ctx, const Csr& A, const float* in, int64_t ld_in, float* out, int64_t ld_out,
          int64_t w, int epi, const float* bias, const float* mask, int64_t ld_mask,
          const Scatter* scat = nullptr);
// Row bins from a host copy of the rowptr.  The upload is asynchronous on
// ctx->stream from A.bins_stage; sync = false leaves the stream unsynchronised
// (the caller guarantees the staging is not rewritten before the copy ran).
void build_bins(rdm_ctx* ctx, Csr& A, const int64_t* rowptr_host, bool sync = true);
// Hot-row panel of the CSR the SpMM streams (A itself, or its hub-core residual):
// device-built reference counts, stable descending order, encoded column stream.
void build_hot(rdm_ctx* ctx, Csr& A);

// gemm.cu
void gemm(rdm_ctx* ctx, int op, const float* X, int64_t ldx, const float* W, int64_t ldw, float* C,
          int64_t ldc, int64_t rows, int64_t k, int64_t m, int epi, const float* bias,
          const float* mask, const Scatter* scat = nullptr);
// C[M x N] = A[M x K] · B with B given as pre-split tf32 hi / lo panels
// Bt[N][K] (K-major, row length ldb; 16-byte aligned), on the tensor cores.
void gemm_tc_panels(rdm_ctx* ctx, const float* A, int64_t lda, const float* bhi, const float* blo,
                    int64_t ldb, float* C, int64_t ldc, int64_t M, int64_t N, int64_t K);
// dense hub core (spmm.cu)
void build_core(rdm_ctx* ctx, Csr& A, const int64_t* rowptr_host, const int32_t* col_host,
                const float* val_host);

// binary hub tiles (hubtiles.cu): host builder (false = values do not factor
// or no tile pays; nothing built) and the per-call product
//   part[item][r][c] = Σ_{tiles of item} T01 · (s ⊙ X[hubs]) (columns < w),
// summed per row block and scaled by s_i in the SpMM epilogue.
bool build_hub_tiles(rdm_ctx* ctx, Csr& A, const int64_t* rowptr_host, const int32_t* col_host,
                     const float* val_host);
// np = pieces of s⊙X: kPiecesI8 = three int8 digits on kind::i8 (fp32-class default), 2 fp16
// (RDM_TILE_PIECES=2), 3 bf16 (RDM_TILE_PIECES=3) or 1 bf16 (RDM_PREC_FAST).
constexpr int kPiecesI8 = 8;     // three int8 digits (23-bit fixed point per column)
constexpr int kPiecesI8x2 = 9;   // two int8 digits (15-bit fixed point): the fast variant
bool hub_tiles_pay(const Core& c, int64_t w, int np);
// int8 tiles in row-block pairs (partials of 256 rows per item, items per pair)
bool tiles_paired();
void hub_tiles_product(rdm_ctx* ctx, const Core& c, const float* X, int64_t ldx, int64_t w,
                       float* part, int64_t ldp, int np);

// hub-core size rule shared by the host (full graph) and device (subgraph) builders
int64_t choose_core_K(const int64_t* bucket, int64_t kmax, const char* force, bool* forced);

// saint.cu — gathers of the full-graph input into a subgraph's slices
void saint_gather(rdm_ctx* ctx, const float* H, int64_t ldh, const int32_t* nodes, int64_t row_lo,
                  int64_t rows, int64_t col_lo, int64_t cols, float* out, int64_t ldo);
void saint_gather_labels(rdm_ctx* ctx, const int32_t* labels, const uint8_t* mask,
                         const int32_t* nodes, int64_t row_lo, int64_t rows, int32_t* lab_out,
                         uint8_t* mask_out);

// runtime.cpp — fused ("p2p") redistribution support
void count_fused_redist(rdm_ctx* ctx, rdm_layout from, int64_t n, int64_t f);
void p2p_barrier(rdm_ctx* ctx);
std::vector<float*> p2p_open(rdm_ctx* ctx, float* mine, std::vector<void*>& opened);

// Round-to-nearest fp32 → tf32 (ties away from zero), used by every 3xTF32 split.
__device__ __forceinline__ float tf32_rn(float x) {
  return __uint_as_float((__float_as_uint(x) + 0x1000u) & 0xFFFFE000u);
}

// redist.cu — pack (row slice → P contiguous blocks, each r x ld_q) and
// unpack (P blocks r x ld_q → row slice).  `blocks[q]` points to block q.
struct BlockTable {
  static constexpr int kMax = 64;
  const float* src[kMax];
  float* dst[kMax];
  int64_t col_lo[kMax];
  int64_t width[kMax];
  int64_t ld[kMax];
};
void pack_rows(rdm_ctx* ctx, const float* row_slice, int64_t ld_row, int64_t rows, int P,
               const BlockTable& t);
void unpack_rows(rdm_ctx* ctx, float* row_slice, int64_t ld_row, int64_t rows, int P,
                 const BlockTable& t);
// bf16 wire of the executor's redistributions under RDM_PREC_FAST (redist.cu):
// pack / unpack with bf16 blocks (the self block stays in fp32, bf16-rounded),
// and the column-slice conversions of the staged side (rows [skip_lo, skip_hi)
// are the self block and are not touched).
void pack_rows_bf16(rdm_ctx* ctx, const float* row_slice, int64_t ld_row, int64_t rows, int P, int self,
                    const BlockTable& t, float* self_dst, int64_t ld_self);
void unpack_rows_bf16(rdm_ctx* ctx, float* row_slice, int64_t ld_row, int64_t rows, int P, int self,
                      const BlockTable& t, const float* self_src, int64_t ld_self);
void narrow_cols(rdm_ctx* ctx, const float* col, int64_t n, int64_t ld, int64_t skip_lo, int64_t skip_hi,
                 void* stage);
void widen_cols(rdm_ctx* ctx, const void* stage, int64_t n, int64_t ld, int64_t skip_lo, int64_t skip_hi,
                float* col);
// Unfused form of a Scatter (producers without a fused epilogue): copies the
// rows x cols slice `src` into the destinations the descriptor names.
void scatter_slice(rdm_ctx* ctx, const float* src, int64_t lds, int64_t rows, int64_t cols,
                   const Scatter& s);

// panels.cpp — R_A < P (§III-E)
void set_graph_panels(rdm_ctx* ctx, int RA, int64_t n, int64_t nnz, const int64_t* rowptr,
                      const int32_t* col, const float* val, int on_host);
void tile_of(int P, int RA, int64_t n, int64_t f, int p, Range* rows, Range* cols, int64_t* ld);
void redistribute_panels(rdm_ctx* ctx, rdm_layout from, const float* const* src, float* const* dst,
                         int64_t n, int64_t f);
void spmm_panels(rdm_ctx* ctx, const float* const* in, float* const* out, int64_t f, int epi,
                 const float* bias, const float* const* mask);
int max_replication(int P, double mem_bytes, double h_all_bytes, double g_bytes);

// misc.cu
void softmax_xent(rdm_ctx* ctx, const float* Z, int64_t ldz, const int32_t* labels,
                  const uint8_t* mask, int64_t rows, int64_t C, const double* n_train, float* G,
                  int64_t ldg, double* loss_partial);
void count_mask(rdm_ctx* ctx, const uint8_t* mask, int64_t rows, double* out);
// out[c] = Σ_r G[r, c] (fp64 accumulation, fixed order), c < cols
void colsum(rdm_ctx* ctx, const float* G, int64_t ldg, int64_t rows, int64_t cols, float* out);
void apply_mask(rdm_ctx* ctx, float* X, int64_t ldx, const float* H, int64_t ldh, int64_t rows,
                int64_t cols);
void sum_slots(rdm_ctx* ctx, float* out, const float* const* parts, int nparts, int64_t count);
void sum_doubles(rdm_ctx* ctx, double* out, const double* const* parts, int nparts);
void finish_loss(rdm_ctx* ctx, const double* sum, const double* n_train, double* loss);
void adam(rdm_ctx* ctx, float* p, const float* g, float* m, float* v, int64_t n, float lr,
          float b1, float b2, float eps, float bc1, float bc2);
void copy_2d(rdm_ctx* ctx, float* dst, int64_t ldd, const float* src, int64_t lds, int64_t rows,
             int64_t cols);

// ---------------------------------------------------------------- transport
// Exchange of the redistribution: for every local slot i and peer q != p,
// send[i][q] (bytes) → slot of q, recv[i][q].
struct Xfer {
  const void* send[BlockTable::kMax];
  void* recv[BlockTable::kMax];
  size_t send_bytes[BlockTable::kMax];
  size_t recv_bytes[BlockTable::kMax];
};
void exchange(rdm_ctx* ctx, std::vector<Xfer>& x);   // x[i] for local slot i
// runtime.cpp — CSR upload / validation (used by rdm_set_graph and the R_A < P panels)
void upload_csr(rdm_ctx* ctx, Csr& A, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col,
                const float* val, bool on_host);
int validate_csr(rdm_ctx* ctx, const int64_t* rowptr, const int32_t* col, int64_t n, int64_t nnz);
void allreduce(rdm_ctx* ctx, float* const* bufs, int64_t count);
void allreduce_d(rdm_ctx* ctx, double* const* bufs, int64_t count);

// redistribution on all local slots (used by rdm_redistribute and the executor)
void redistribute(rdm_ctx* ctx, rdm_layout from, const float* const* src, float* const* dst,
                  int64_t n, int64_t f, bool bf16_wire = false);

// ------------------------------------------------------------------- plan
int64_t config_to_id(const rdm_config& c);
rdm_config config_from_id(int L, int64_t id);
void model_costs(int L, const int64_t* f, int need_input_grad, const rdm_config& c, int64_t* comm,
                 int64_t* sparse);

}  // namespace rdm
