/* rdm.h — C ABI of the B200-native GNN-RDM hot path.
 *
 * GNN-RDM (Kurt, Yan, Sukumaran-Rajam, Pandey, Sadayappan, IPDPS'23,
 * "Communication Optimization for Distributed Execution of Graph Neural
 * Networks"); citations are PAPER.md line numbers "L<n>" with the section,
 * equation or table they fall in.
 *
 * The method: a full-batch GCN layer Z^l = Aᵀ H^{l-1} W^l, H^l = σ(Z^l)
 * (eq. 1-2) and its backward (eq. 3-4) distributed over P
 * processes with NO communication inside the products:
 *   - SpMM  Out = A·In    with A replicated, In/Out column ("vertically")
 *     sliced  (§III-A, Fig. 2a);
 *   - GEMM  Out = In·W    with W replicated, In/Out row ("horizontally")
 *     sliced  (Fig. 2b);
 *   - an all-to-all personalized redistribution between the two layouts is
 *     the only bulk communication (§III-D; Fig. 7);
 *   - the order (AᵀH)W vs Aᵀ(HW) is chosen per layer, forward and backward,
 *     by a redistribution-volume / SpMM-op-count model (§IV, Tables II-IV,
 *     Pareto set Table VI).
 *
 * Conventions for every entry point
 * ---------------------------------
 *  * Return value: an rdm_status.  Nothing is thrown across the ABI.  On a
 *    non-RDM_OK status, rdm_last_error(ctx) returns a human-readable reason
 *    (thread-unsafe; one ctx per thread).  Arguments are validated
 *    synchronously (RDM_ERR_ARG).  Kernel-launch errors are reported
 *    immediately (RDM_ERR_CUDA); asynchronous device faults surface at
 *    rdm_sync() or the next call.  After an NCCL failure the communicator is
 *    aborted and every later call on the ctx returns RDM_ERR_STATE.
 *  * Asynchrony: every call that takes a ctx enqueues its work on the ctx's
 *    CUDA stream and returns without synchronising, except rdm_set_graph,
 *    rdm_gcn_create/set_input (setup, synchronous) and the pure host
 *    functions (rdm_partition, rdm_config_*, rdm_select_config).
 *  * Memory: all float / index buffers passed to compute entry points are
 *    CUDA device memory on the ctx's device unless a parameter says
 *    otherwise (`on_host`).  The caller owns every buffer it passes; the
 *    library owns the device CSR copy, the row bins, the pack/recv
 *    workspace, the NCCL communicator and the activation workspace of an
 *    rdm_gcn.  Nothing the caller passed is freed by the library.
 *  * Dense layout: row-major fp32 with a leading dimension `ld` (elements)
 *    that is a multiple of 4 and 16-byte aligned base pointers; columns
 *    [width, ld) are padding and must hold zeros on input (outputs keep them
 *    zero).  rdm_partition() returns the ld the library expects.
 *  * Ranks: a ctx is either ONE rank of a P-process NCCL job (one process per
 *    GPU) or, with rank == RDM_ALL_RANKS, a "virtual group" holding all P
 *    ranks in this process on one device, whose all-to-all is a device copy
 *    (used to exercise the P>1 partitions, pack/unpack and executor on a
 *    single GPU).  Collective entry points take one pointer per LOCAL rank
 *    (1 for an NCCL rank, P for a virtual group, local slot i = rank i).
 *  * Collective entry points (rdm_redistribute, rdm_allreduce_sum,
 *    rdm_gcn_forward, rdm_gcn_backward, rdm_gcn_set_input) must be called
 *    by every rank in the same order.
 */
#ifndef RDM_H
#define RDM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define RDM_ABI_VERSION 1
#define RDM_ALL_RANKS (-1)
#define RDM_MAX_LAYERS 8
#define RDM_UNIQUE_ID_BYTES 128

typedef struct rdm_ctx rdm_ctx; /* one per process (= one per GPU), or one virtual group */
typedef struct rdm_gcn rdm_gcn; /* a GCN model instance: config + activation workspace */

typedef enum {
  RDM_OK = 0,
  RDM_ERR_ARG = 1,         /* invalid argument / size / layout; nothing enqueued            */
  RDM_ERR_CUDA = 2,        /* CUDA runtime or launch error                                  */
  RDM_ERR_NCCL = 3,        /* NCCL error; the communicator has been aborted                 */
  RDM_ERR_OOM = 4,         /* device allocation failed (e.g. A does not fit: R_A < P, L148) */
  RDM_ERR_UNSUPPORTED = 5, /* valid request this build does not implement                   */
  RDM_ERR_STATE = 6        /* ctx poisoned by an earlier NCCL/CUDA fault, or call order     */
} rdm_status;

/* Row-sliced ("horizontal", Fig. 2b) or column-sliced ("vertical", Fig. 2a). */
typedef enum { RDM_ROW = 0, RDM_COL = 1 } rdm_layout;

/* Fused epilogues (bit set).  BIAS: out[:, c] += bias[c] (reading R8);
 * RELU: σ = ReLU (reading R4); MASK: out ⊙= 1[mask > 0], the Hadamard with
 * σ'(Z^{l-1}) of eq. (3), given H^{l-1} = ReLU(Z^{l-1}) in the same layout. */
enum { RDM_EPI_NONE = 0, RDM_EPI_BIAS = 1, RDM_EPI_RELU = 2, RDM_EPI_MASK = 4 };

/* GEMM forms (eq. 1, 3, 4).  rows = local row count, W is k x m:
 *   NN: C[rows x m] = X[rows x k] · W          (forward, Z = T W or T = H W)
 *   NT: C[rows x k] = X[rows x m] · Wᵀ         (backward data, A G Wᵀ)
 *   TN: C[k x m]    = X[rows x k]ᵀ · U[rows x m] (weight gradient, eq. 4) */
enum { RDM_GEMM_NN = 0, RDM_GEMM_NT = 1, RDM_GEMM_TN = 2 };

/* One configuration (Table IV): for each layer l = 1..L (index
 * l-1), 1 = GEMM first ("D", dense first), 0 = SpMM first ("S").  The
 * integer ID of a config puts bits MSB→LSB as [bwd L … bwd 1, fwd 1 … fwd L]
 * (for L = 2: ID = 8·bwdL2 + 4·bwdL1 + 2·fwdL1 + fwdL2; ID 10 = the
 * dense-sparse-dense-sparse path of Fig. 4). */
typedef struct {
  int L;
  uint8_t fwd_D[RDM_MAX_LAYERS];
  uint8_t bwd_D[RDM_MAX_LAYERS];
} rdm_config;

/* Flags for rdm_gcn_create. */
enum {
  RDM_GCN_INPUT_GRAD = 1, /* also compute G^0 = A G^1 (W^1)ᵀ (Fig. 4 output; reading R2) —
                             required for costs to match Table IV                       */
  RDM_GCN_BIAS = 2,       /* Z^l = Â H^{l-1} W^l + 1 (b^l)ᵀ before σ (reading R8): the bias
                             is fused into the epilogue of Z^l's producer (the SpMM or the
                             GEMM, whichever runs last for the layer's config); the backward
                             pass adds db^l = 1ᵀ G^l (deterministic fp64 column sums of the
                             masked G^l in whatever layout it is resident, all-reduced with
                             Y^l).  rdm_gcn_forward/backward then require b / db.          */
  RDM_GCN_PANELS = 4,     /* R_A < P (§III-E): run on the row panels installed by
                             rdm_set_graph_panels (a symmetric A) instead of the replicated
                             graph; column-layout tensors are tiles (rdm_partition_tile),
                             SpMMs broadcast input tiles inside column groups, redistributions
                             stay inside panel groups; RDM_TRANSPORT_P2P fusion is not used */
  RDM_GCN_LOW_MEMORY = 8  /* liveness-based workspace: buffers of the same shape whose lifetimes
                             within an epoch do not overlap share one allocation (first fit,
                             largest first).  Results are identical; rdm_gcn_tensor returns
                             RDM_ERR_STATE for a tensor whose memory a later step reuses.  For
                             the stress shapes (papers100M-shaped at P = 8, SURVEY App. B:
                             "~70 GB/GPU of live tensors with liveness-based reuse")      */
};

/* Tensors exposed by rdm_gcn_tensor (for parity tests / inspection). */
enum {
  RDM_T_H = 0,    /* H^l, l = 0..L-1                                   */
  RDM_T_Z = 1,    /* logits Z^L (layer argument ignored)               */
  RDM_T_G = 2,    /* G^l = ∂ℓ/∂Z^l, l = 0..L (G^0 = ∂ℓ/∂H^0)           */
  RDM_T_MEMO = 3, /* T_l = Aᵀ H^{l-1}, row-sliced, S-first layers (L134) */
  RDM_T_DWP = 4   /* this rank's partial Y^l before the all-reduce     */
};

/* Per-phase timers (Fig. 12 analogue: communication vs computation). */
enum {
  RDM_PH_SPMM = 0,
  RDM_PH_GEMM = 1,
  RDM_PH_PACK = 2,      /* pack + unpack kernels of the redistribution  */
  RDM_PH_A2A = 3,       /* NCCL grouped send/recv (or virtual copies)    */
  RDM_PH_LOSS = 4,
  RDM_PH_ALLREDUCE = 5, /* Y^l / loss all-reduce                         */
  RDM_PH_ADAM = 6,
  RDM_PH_OTHER = 7,
  RDM_PH_SAMPLE = 8,    /* GraphSAINT sampler + induced-subgraph build    */
  RDM_PH_COUNT = 9
};

typedef struct {
  int64_t a2a_calls;          /* redistributions executed                                    */
  int64_t a2a_elems_payload;  /* elements crossing ranks (exact partition, no padding)       */
  int64_t a2a_bytes_wire;     /* bytes handed to the transport for other ranks (incl. pad)   */
  int64_t a2a_width_units;    /* Σ widths f of redistributions = the model's comm units      */
  int64_t spmm_calls;
  int64_t spmm_nnz_cols;      /* Σ nnz · w over SpMM calls (sparse ops, L142)                 */
  int64_t spmm_width_units;   /* Σ full widths f of SpMM steps = the model's sparse units    */
  int64_t gemm_calls;
  int64_t gemm_flops;
  int64_t allreduce_bytes;
  int64_t kernel_launches;    /* kernels this library launched                               */
  int64_t bcast_elems;        /* R_A < P: elements of input tiles broadcast to other ranks   */
} rdm_counters;

/* ---------------------------------------------------------------- context */

/* ncclGetUniqueId into id[RDM_UNIQUE_ID_BYTES]; rank 0 calls it and the caller
 * broadcasts the bytes (e.g. with torch.distributed). */
rdm_status rdm_get_unique_id(void* id);

/* Create a context on CUDA device `device`, enqueuing on `cuda_stream`
 * (cudaStream_t; NULL = the legacy default stream).
 *   world == 1                  : single process, no NCCL.
 *   0 <= rank < world, world > 1: one rank of an NCCL job; `nccl_unique_id`
 *                                 (RDM_UNIQUE_ID_BYTES) from rdm_get_unique_id.
 *   rank == RDM_ALL_RANKS       : virtual group of `world` ranks in-process.
 * Errors: RDM_ERR_ARG (bad rank/world/device), RDM_ERR_CUDA, RDM_ERR_NCCL. */
rdm_status rdm_init(rdm_ctx** ctx, int rank, int world, const void* nccl_unique_id, int device,
                    void* cuda_stream);
/* One-rank emulation of a P-rank job (measurement of the stress shapes, e.g.
 * BASELINE configs[4], papers100M-shaped at P = 8, on a single GPU): a ctx
 * that is rank `rank` of `world` ranks with NO peers and no NCCL.  It holds
 * exactly that rank's partitions (row slice rows_p x f, column slices
 * N x w_p, its staging buffers) and runs exactly that rank's SpMMs, GEMMs,
 * pack/unpack, loss and Adam at the P-rank shapes; every exchange and
 * all-reduce is skipped (nothing crosses a link: the received blocks keep
 * their previous contents and the counters still count the traffic a real
 * rank would move).  For timing and memory measurement only — the numerical
 * results are NOT those of the P-rank job.  RDM_TRANSPORT_P2P is refused
 * (RDM_ERR_UNSUPPORTED).  Errors: RDM_ERR_ARG (world < 2, rank), RDM_ERR_CUDA. */
rdm_status rdm_init_emulated(rdm_ctx** ctx, int rank, int world, int device, void* cuda_stream);
int rdm_is_emulated(const rdm_ctx* ctx);
/* The NCCL communicator behind the ctx (one rank of an NCCL job): NCCL
 * version code, ncclCommCount, ncclCommUserRank, ncclCommCuDevice.  Without a
 * communicator (world 1, virtual group, emulated rank) comm_ranks = 0 and
 * comm_rank = comm_device = -1.  Any output pointer may be NULL. */
rdm_status rdm_comm_info(rdm_ctx* ctx, int* nccl_version, int* comm_ranks, int* comm_rank,
                         int* comm_device);
rdm_status rdm_finalize(rdm_ctx* ctx);
const char* rdm_last_error(const rdm_ctx* ctx);
/* Block until the ctx's stream is idle; surfaces asynchronous CUDA/NCCL faults. */
rdm_status rdm_sync(rdm_ctx* ctx);
rdm_status rdm_set_stream(rdm_ctx* ctx, void* cuda_stream);

/* Transport of the GCN executor's redistributions (§III-D; SURVEY
 * §8(e) "Phase 2"):
 *   RDM_TRANSPORT_NCCL (default): pack → NCCL grouped send/recv → unpack.
 *   RDM_TRANSPORT_P2P: a redistribution whose source was produced by the
 *     step right before it is fused into that producer: the GEMM (row → col)
 *     or SpMM (col → row) epilogue stores every output element straight into
 *     its owner's destination slice — the other slots' buffers in a virtual
 *     group, CUDA-IPC-mapped peer memory over NVLink for NCCL ranks (fenced
 *     by two one-word NCCL all-reduces around the producer).  Unfused
 *     redistributions keep the NCCL path.  Results are bit-identical to the
 *     default (pure data movement); counters count the same logical traffic.
 * Takes effect for GCN instances created afterwards.  The environment
 * variable RDM_P2P=1 selects P2P at rdm_init.  Errors: RDM_ERR_ARG. */
enum { RDM_TRANSPORT_NCCL = 0, RDM_TRANSPORT_P2P = 1 };
rdm_status rdm_set_transport(rdm_ctx* ctx, int transport);
int rdm_get_transport(const rdm_ctx* ctx);

/* Arithmetic variant of the operators (BASELINE
 * north_star: "2e-2 if a bf16 GEMM variant is enabled"):
 *   RDM_PREC_FP32 (default): fp32 storage and accumulation, GEMMs in 3xTF32
 *     on the tensor cores — the 1e-4 parity gate.
 *   RDM_PREC_FAST: every rdm_spmm rounds its input column slice to bf16
 *     (round-to-nearest-even) once per call and gathers the bf16 rows
 *     (half the L2/HBM gather bytes), accumulating in fp32; the binary hub
 *     tiles multiply one bf16 piece of s⊙X (fp32: two column-scaled fp16 or three bf16 pieces); every rdm_gemm
 *     NN / NT runs on kind::f16 with bf16 operands (X rounded to nearest even
 *     as it is staged, W as bf16 panels; fp32 accumulation; RDM_F16_GEMM=0
 *     keeps one tf32 MMA per k step), TN issues one tf32 MMA per k step
 *     instead of 3xTF32.  Inside rdm_gcn_forward /
 *     backward the row → column redistributions (whose destination is an
 *     SpMM input, rounded to bf16 by the variant anyway) carry bf16 on the
 *     wire (half their bytes; each moved value, the rank's own block included,
 *     rounded once); column → row moves stay fp32.  Outputs, gradients and the
 *     loss stay fp32 in the caller's buffers; the public rdm_redistribute
 *     stays bit-exact fp32.
 *     Parity gate 2e-2 (max relative error per tensor, reading R26).
 * Applies to every later call on the ctx (the executor included).
 * Errors: RDM_ERR_ARG (unknown value). */
enum { RDM_PREC_FP32 = 0, RDM_PREC_FAST = 1 };
rdm_status rdm_set_precision(rdm_ctx* ctx, int precision);
int rdm_get_precision(const rdm_ctx* ctx);

int rdm_world(const rdm_ctx* ctx);
int rdm_num_local(const rdm_ctx* ctx);            /* local rank slots (1 or world)  */
int rdm_local_rank(const rdm_ctx* ctx, int slot); /* global rank of local slot      */

/* Partition (reading R11; the paper draws even halves, Fig. 5/7):
 *   RDM_ROW: rows [lo, hi) of n, lo = ⌊rank·n/world⌋; ld = roundup(f, 4)
 *   RDM_COL: cols [lo, hi) of f in 4-float granules g = ⌈f/4⌉,
 *            lo = min(f, 4·⌊rank·g/world⌋); ld = roundup(hi − lo, 4)
 * Pure host function. */
rdm_status rdm_partition(int world, rdm_layout layout, int64_t n, int64_t f, int rank,
                         int64_t* lo, int64_t* hi, int64_t* ld);

/* ------------------------------------------------------------------ graph */

/* Install the replicated sparse adjacency A (N x N CSR: int64 rowptr[n+1],
 * int32 col[nnz], fp32 val[nnz]) on every local rank — R_A = P full
 * replication (§III-E).  Values are used as given (the GCN
 * normalization is the caller's, L255).  `symmetric` != 0 promises A = Aᵀ
 * (one CSR serves eq. 1's Aᵀ and eq. 3-4's A, reading R3); otherwise the
 * transpose is built.  `on_host` != 0: pointers are host memory.  Validates
 * rowptr monotonicity and column range (RDM_ERR_ARG) and builds the row
 * bins (light rows warp-per-row, heavy rows split into fixed nnz segments).
 * RDM_ERR_OOM if A does not fit (R_A < P is not supported).  Synchronous. */
rdm_status rdm_set_graph(rdm_ctx* ctx, int64_t n, int64_t nnz, const int64_t* rowptr,
                         const int32_t* col, const float* val, int symmetric, int on_host);

/* What rdm_set_graph built: row bins (light rows warp-per-row, heavy rows in
 * 2048-nnz segments) and, for symmetric graphs with a dense block of
 * high-degree vertices, the "hub core": the K x K block A[hubs, hubs] (K a
 * multiple of 128, core_nnz entries) held dense and multiplied on the tensor
 * cores, the other entries in a residual CSR (core_K = 0: no core).
 * When every value of the hub region factors as a_ij = r_i c_j (a rank-1
 * scaling of the 0/1 pattern: the GCN normalization D^-1/2 (A+I) D^-1/2, the
 * row-normalized D^-1 (A+I), all ones, …; r and c found by a walk over the
 * moved entries and checked entry by entry to 2^-21 relative) the core is
 * instead a set of "binary hub tiles": the tile_ranks highest-degree
 * vertices' block cut into 128 x 128 rank blocks, the n_tiles blocks dense
 * enough to pay stored as bits and multiplied on the tensor cores against
 * c ⊙ X (three int8 digits of a per-column 23-bit fixed point on kind::i8 by
 * default), r applied in the residual SpMM's epilogue (core_K = 0,
 * core_nnz = entries moved). */
typedef struct {
  int64_t n, nnz;
  int64_t n_light_rows, n_heavy_rows, n_segments, max_degree;
  int64_t core_K, core_nnz;
  int symmetric;
  int64_t tile_ranks, n_tiles, n_tile_items;
} rdm_graph_info;
rdm_status rdm_get_graph_info(const rdm_ctx* ctx, rdm_graph_info* out);

/* --------------------------------------------------- communication-free ops */

/* Communication-free SpMM on one column slice (Fig. 2a):
 *   out[N x w] = op(A) · in[N x w],  op(A) = Aᵀ if transpose (eq. 1) else A
 * (eq. 3-4).  in/out: row-major, leading dims ld_in/ld_out (multiples of 4,
 * ≥ w).  Epilogue bits RDM_EPI_*: bias[w] (device) added, then ReLU, then
 * ⊙ 1[mask > 0] with mask[N x w] at leading dim ld_mask.  Local: no
 * communication.  Deterministic (fixed summation order, no float atomics). */
rdm_status rdm_spmm(rdm_ctx* ctx, int transpose, const float* in, int64_t ld_in, float* out,
                    int64_t ld_out, int64_t w, int epilogue, const float* bias, const float* mask,
                    int64_t ld_mask);

/* Communication-free GEMM on row slices (Fig. 2b), fp32-accurate.
 * op = RDM_GEMM_NN / NT / TN (see above); X at leading dim ldx, W k x m
 * contiguous (ldw = m) for NN/NT; for TN the second operand U is rows x m at
 * leading dim ldw.  C at leading dim ldc.  Epilogue (NN/NT only): BIAS, RELU,
 * MASK (mask at leading dim ldc).  Local: no communication. */
rdm_status rdm_gemm(rdm_ctx* ctx, int op, const float* X, int64_t ldx, const float* W, int64_t ldw,
                    float* C, int64_t ldc, int64_t rows, int64_t k, int64_t m, int epilogue,
                    const float* bias, const float* mask);

/* ------------------------------------------------------------- collectives */

/* All-to-all personalized redistribution of an N x f matrix between the
 * row-sliced and column-sliced layouts (§III-D, Fig. 7: divide
 * into P chunks → exchange → merge).  from = RDM_ROW: src[i] is local slot
 * i's row slice (rows_p x ld_row), dst[i] its column slice (N x ld_col_p);
 * from = RDM_COL the reverse.  Pure data movement: bit-exact.  Moves
 * Σ_{p≠q} rows·cols ≈ (P−1)/P·N·f elements in total (L142).  P = 1: copies
 * src to dst if they differ (the two layouts coincide). */
rdm_status rdm_redistribute(rdm_ctx* ctx, rdm_layout from, const float* const* src,
                            float* const* dst, int64_t n, int64_t f);

/* Exchange plan of one redistribution for `rank` (pure host function), per
 * peer q (arrays of `world` entries, element units): the rank sends
 * send_elems[q] floats starting at send_off[q] and receives recv_elems[q]
 * floats at recv_off[q].  from = RDM_ROW: sends from the packed staging
 * buffer (blocks rows_p x ld_q in q order), receives straight into its
 * column slice; from = RDM_COL: sends straight from its column slice,
 * receives into the staging buffer (then merged).  Self entries are 0 (the
 * self block is copied on-device).  Wire blocks are ld-padded (rdm.h). */
rdm_status rdm_redist_plan(int world, int rank, rdm_layout from, int64_t n, int64_t f,
                           int64_t* send_off, int64_t* send_elems, int64_t* recv_off,
                           int64_t* recv_elems);

/* -------------------------------------------- partial replication, R_A < P */
/* §III-E (L146-167, Fig. 6), Tables II/III "Comm. (R_A < P)" rows, §IV-A.4
 * (L214-216); SURVEY §8(f) NEXT-4.  The P ranks form a grid of P/R_A row
 * panels x R_A column groups, rank p = i·R_A + j.  Row panel i of the
 * adjacency (rows row_range(N, P/R_A, i) — ⌊i·N·R_A/P⌋ … — all N columns) is
 * stored on the R_A ranks of panel group i: R_A copies of A in total instead
 * of P.  Dense SpMM operands use the TILE layout: rank (i, j) holds panel i's
 * rows x the column range of RDM_COL partitioned over R_A (rdm_partition_tile).
 *
 * rdm_set_graph_panels: install the panels this process needs (1 for an NCCL
 *   rank, P/R_A for a virtual group).  The matrix is used as given (pass Aᵀ
 *   for eq. 1 on a directed graph).  R_A must divide P.  Synchronous.  Errors:
 *   RDM_ERR_ARG (R_A, CSR), RDM_ERR_OOM.  Independent of rdm_set_graph.
 * rdm_partition_tile: rank's tile (pure host function): rows [row_lo, row_hi),
 *   columns [col_lo, col_hi), leading dim ld = roundup4(col_hi − col_lo).
 * rdm_redistribute_panels: row slices (rdm_partition RDM_ROW) ↔ tiles, an
 *   all-to-all inside every panel group: (R_A−1)/R_A·N·f elements in total
 *   (L214).  from = RDM_ROW: src row slices → dst tiles; RDM_COL: tiles →
 *   row slices.  Collective, bit-exact.
 * rdm_spmm_panels: out_tile = A[panel rows, :] · In[:, tile columns] (Fig. 6):
 *   each rank broadcasts its input tile to the other P/R_A − 1 ranks of its
 *   column group ((P/R_A − 1)·N·f elements per call, L152/L216, counted in
 *   rdm_counters.bcast_elems), then multiplies its row panel by the
 *   assembled N x w_j slice (the rdm_spmm kernels, honouring
 *   rdm_set_precision).  Epilogue bits as rdm_spmm; bias: f floats (device,
 *   replicated) or NULL; mask: one tile per local slot or NULL.  Collective.
 * rdm_max_replication: L160-167 R_A = P·(M − H_all)/G capped at P; the
 *   largest divisor of P not above it (reading R36); 0 if A does not fit in
 *   the aggregate memory.  Pure host function. */
rdm_status rdm_set_graph_panels(rdm_ctx* ctx, int R_A, int64_t n, int64_t nnz, const int64_t* rowptr,
                                const int32_t* col, const float* vals, int on_host);
rdm_status rdm_partition_tile(int world, int R_A, int64_t n, int64_t f, int rank, int64_t* row_lo,
                              int64_t* row_hi, int64_t* col_lo, int64_t* col_hi, int64_t* ld);
rdm_status rdm_redistribute_panels(rdm_ctx* ctx, rdm_layout from, const float* const* src,
                                   float* const* dst, int64_t n, int64_t f);
rdm_status rdm_spmm_panels(rdm_ctx* ctx, const float* const* in_tiles, float* const* out_tiles,
                           int64_t f, int epilogue, const float* bias, const float* const* mask_tiles);
int rdm_max_replication(int world, double mem_bytes_per_gpu, double h_all_bytes_per_gpu,
                        double graph_bytes);
/* Configuration choice at R_A < P (reading R35): each config's elements moved
 * per epoch = N·[(R_A−1)/R_A·comm_units + (P/R_A−1)·sparse_units] (Tables
 * II/III R_A rows); Pareto-optimal configs in (elements, sparse units) into
 * pareto_ids (*n_pareto: capacity in, count out) and the pick of the same
 * B200 time model as rdm_select_config.  R_A = P reproduces rdm_select_config's
 * front.  Pure host function.  Errors: RDM_ERR_ARG (R_A ∤ P, sizes). */
rdm_status rdm_select_config_ra(int L, const int64_t* f, int64_t n, int64_t nnz, int P, int R_A,
                                int need_input_grad, int64_t* pareto_ids, int* n_pareto,
                                int64_t* chosen_id, double* comm_elems, int64_t* sparse_units);

/* In-place sum over all ranks of count floats per local slot (weight-gradient
 * reduction, reading R16).  Virtual group: every slot receives the sum. */
rdm_status rdm_allreduce_sum(rdm_ctx* ctx, float* const* bufs, int64_t count);

/* ----------------------------------------------------- cost model / selector */

/* Decode / encode a configuration ID (see rdm_config). */
rdm_status rdm_config_from_id(int L, int64_t id, rdm_config* out);
int64_t rdm_config_to_id(const rdm_config* cfg);

/* The paper's model cost of one configuration (§IV-A/B, Tables II-IV):
 * comm_units = Σ redistribution widths (units of (P−1)/P·N elements),
 * sparse_units = Σ SpMM widths (units of nnz FMAs).  f has L+1 entries.
 * need_input_grad must be 1 for Table IV's costs (G^0 is an output, Fig. 4).
 * Pure host function. */
rdm_status rdm_config_costs(int L, const int64_t* f, int need_input_grad, int64_t id,
                            int64_t* comm_units, int64_t* sparse_units);

/* Enumerate the 4^L configurations, keep the Pareto-optimal ones in
 * (comm, sparse) (L31, L224; ties kept, reading R23) into pareto_ids
 * (*n_pareto: capacity in, count out), and pick one (reading R23): the
 * minimum of a B200-calibrated time model t = comm·(P−1)/P·N·4 B / B_link +
 * Σ_spmm (8·nnz + 8·N·w/P) / B_hbm, ties → fewer SpMM width → lower ID.
 * P = 1: comm is free, so the pick is the minimum sparse cost (reading R24).
 * Pure host function. */
rdm_status rdm_select_config(int L, const int64_t* f, int64_t n, int64_t nnz, int P,
                             int need_input_grad, int64_t* pareto_ids, int* n_pareto,
                             int64_t* chosen_id, int64_t* comm_units, int64_t* sparse_units);

/* -------------------------------------------------------------------- GCN */

/* Create a GCN instance with L layers of widths f[0..L] using configuration
 * cfg, and allocate its activation workspace on every local rank.  Requires
 * rdm_set_graph.  flags: RDM_GCN_*.  Synchronous. */
rdm_status rdm_gcn_create(rdm_ctx* ctx, int L, const int64_t* f, const rdm_config* cfg, int flags,
                          rdm_gcn** out);
rdm_status rdm_gcn_destroy(rdm_gcn* g);

/* Per local slot i: H0_row[i] = the rank's row slice of H^0 (rows_p x f0,
 * dense, ld = f0), labels_row[i] (int32, rows_p), mask_row[i] (uint8 train
 * mask, rows_p; NULL = all rows).  Builds H^0 in every layout the config
 * reads (the model charges nothing for H^0's layout, reading R12) and n_train
 * (global).  Collective.
 * `on_host` == 0: device pointers, applied on the ctx stream immediately.
 * `on_host` != 0: host pointers (pinned): ASYNCHRONOUS and double-buffered —
 * the H2D copy is enqueued on a private copy stream into staging buffers
 * (after the previously staged input was consumed) and the next
 * rdm_gcn_forward consumes it, so the copy of step i+1's input overlaps step
 * i's compute.  The host buffers must stay unmodified until that forward has
 * completed (rdm_sync). */
rdm_status rdm_gcn_set_input(rdm_gcn* g, const float* const* H0_row,
                             const int32_t* const* labels_row, const uint8_t* const* mask_row,
                             int on_host);

/* Forward pass of all layers + loss (eq. 1-2; loss L206, reading R5).  W[l]
 * (l = 0..L-1) = W^{l+1}, f_l x f_{l+1} row-major, replicated (one copy per
 * process).  b: with RDM_GCN_BIAS, b[l] = b^{l+1} (f_{l+1} floats, device,
 * replicated), RDM_ERR_ARG if b or any b[l] is null; ignored otherwise (may
 * be null).  loss_dev: device double, receives the global mean loss.
 * Collective. */
rdm_status rdm_gcn_forward(rdm_gcn* g, const float* const* W, const float* const* b,
                           double* loss_dev);

/* Backward pass (eq. 3-4) with fwd→bwd memo reuse (§III-C):
 * dW[l] receives Y^{l+1}, all-reduced over ranks (one copy per process);
 * with RDM_GCN_BIAS, db[l] (f_{l+1} floats, device) receives db^{l+1} =
 * 1ᵀ G^{l+1}, all-reduced likewise (RDM_ERR_ARG if null); db is ignored
 * otherwise.  Collective. */
rdm_status rdm_gcn_backward(rdm_gcn* g, const float* const* W, float* const* dW, float* const* db);

/* What the executor will run for this instance (per epoch, per rank):
 *   model_*  : the paper's cost of the config (rdm_config_costs);
 *   plan_*   : the units the executor actually issues — redistribution widths
 *              (incl. `plan_hidden_comm_units`, transfers the paper's model
 *              does not charge, e.g. the Hadamard operand of IDs 6/9,
 *              reading R15) and SpMM widths; at P = 1 no redistribution runs.
 *   a2a_elems: exact elements crossing ranks per epoch summed over all ranks
 *              (Σ over redistributions of Σ_{p≠q} rows·cols, no padding). */
typedef struct {
  int64_t model_comm_units, model_sparse_units;
  int64_t plan_comm_units, plan_hidden_comm_units, plan_sparse_units;
  int64_t a2a_elems;
  int n_fwd_steps, n_bwd_steps;
  int64_t workspace_bytes; /* activation workspace per process (rdm_plan_info: of rank 0,
                              honouring RDM_GCN_LOW_MEMORY in flags)                      */
} rdm_gcn_info;
rdm_status rdm_gcn_get_info(const rdm_gcn* g, rdm_gcn_info* out);
/* Human-readable step list (forward then backward) into buf[cap]. */
rdm_status rdm_gcn_describe(const rdm_gcn* g, char* buf, size_t cap);
/* The same plan for a hypothetical instance (pure host function, no ctx):
 * L layers, widths f[0..L], config cfg, P ranks, N vertices, RDM_GCN_* flags.
 * `desc` (may be NULL) receives the step list. */
rdm_status rdm_plan_info(int L, const int64_t* f, const rdm_config* cfg, int P, int64_t n,
                         int flags, rdm_gcn_info* out, char* desc, size_t cap);

/* Device pointer + shape of an internal tensor of local slot `slot` in
 * `layout` (RDM_ERR_ARG if that layout is not resident). */
rdm_status rdm_gcn_tensor(rdm_gcn* g, int which, int layer, int slot, rdm_layout layout,
                          const float** ptr, int64_t* rows, int64_t* cols, int64_t* ld);

/* ------------------------------------------------------ GraphSAINT-RDM */

/* Sampling-based training (§III-F, §V-C): "graph-sampling
 * to create independently processed subgraphs" (GraphSAINT [17]); "each
 * subgraph is parallelized using our RDM scheme" (L388) and the weights are
 * updated after each subgraph (L390).  "A random generated seed can be
 * passed to all processes and each process can generate its sparse mask
 * individually" (L173): every rank samples the SAME subgraph from the shared
 * seed — no communication.
 *
 * Sampler (readings R31-R34): GraphSAINT random-walk sampler on
 * the installed graph (rdm_set_graph; walks follow its stored CSR entries,
 * self loops included).  For subgraph `it`, with key = splitmix64(seed +
 * it·0x9E3779B97F4A7C15) and u(i, j) = splitmix64(key ^ (i << 8 | j)):
 * root i (0 ≤ i < roots) is u(i, 0) mod N; step j = 1..walk_len moves from v
 * to col[rowptr[v] + u(i, j) mod deg(v)].  The node set is the sorted set of
 * visited vertices (new id = rank in that order).  The subgraph is the
 * induced one, Â_s[i][j] = 1/sqrt(d_i·d_j) for every stored entry (v_i, v_j)
 * with both ends sampled, d_i = entries of row i kept (GCN normalisation of
 * the induced graph, entries in the original row order), computed as
 * (float)(1.0 / sqrt((double)d_i·d_j)).
 * Requires a symmetric graph.  walk_len ≤ 255.  The sampler's GCN instances
 * hold capacity for n_cap = min(N, roots·(walk_len + 1)) vertices. */
typedef struct rdm_saint rdm_saint;
rdm_status rdm_saint_create(rdm_ctx* ctx, int64_t roots, int walk_len, uint64_t seed,
                            rdm_saint** out);
rdm_status rdm_saint_destroy(rdm_saint* s);
/* Sample subgraph number `iteration` and build its CSR on the device (GPU
 * random walks, vertex compaction, induced-subgraph extraction, row bins).
 * Returns its vertex and entry counts.  Synchronises the ctx stream (the
 * host needs the sizes for the executor's launch shapes). */
rdm_status rdm_saint_sample(rdm_saint* s, int64_t iteration, int64_t* n_sub, int64_t* nnz_sub);
/* Make the ctx's stream wait for the sampler's latest subgraph build (which
 * runs on the sampler's own stream and double-buffers its subgraphs, so a
 * sample can overlap the training of the previous subgraph).  The executor
 * does this itself when it switches subgraphs; for timing brackets. */
rdm_status rdm_saint_wait(rdm_saint* s);
/* Device pointers to the current subgraph: nodes[n] (int32 original ids,
 * ascending), rowptr[n+1] (int64), col[nnz] (int32 new ids), val[nnz]. */
rdm_status rdm_saint_subgraph(const rdm_saint* s, const int32_t** nodes, const int64_t** rowptr,
                              const int32_t** col, const float** val, int64_t* n, int64_t* nnz);
/* A GCN instance (as rdm_gcn_create) whose graph is the sampler's current
 * subgraph; forward/backward/adam as for any rdm_gcn.  Destroy the GCN
 * before the sampler. */
rdm_status rdm_saint_gcn_create(rdm_saint* s, int L, const int64_t* f, const rdm_config* cfg,
                                int flags, rdm_gcn** out);
/* Input of the current subgraph for every local slot, gathered on the device
 * from the FULL-graph arrays every rank holds (H0_full N x f0 at leading
 * dim ld_h, labels_full[N], mask_full[N] or NULL = all): H^0 row and column
 * slices, labels, mask and the subgraph's training count.  No communication.
 * Call after each rdm_saint_sample, before rdm_gcn_forward. */
rdm_status rdm_saint_set_input(rdm_gcn* g, const float* H0_full, int64_t ld_h,
                               const int32_t* labels_full, const uint8_t* mask_full);

/* Adam (PyTorch semantics, no weight decay; L297 lr = 0.01) on `count`
 * replicated parameter arrays of sizes[i] floats; step ≥ 1. */
rdm_status rdm_adam_step(rdm_ctx* ctx, int count, float* const* params, const float* const* grads,
                         float* const* m, float* const* v, const int64_t* sizes, float lr,
                         float beta1, float beta2, float eps, int step);

/* -------------------------------------------------------- instrumentation */
rdm_status rdm_get_counters(const rdm_ctx* ctx, rdm_counters* out);
rdm_status rdm_reset_counters(rdm_ctx* ctx);
/* Enable per-phase CUDA-event timing on the ctx stream (small overhead). */
rdm_status rdm_set_timing(rdm_ctx* ctx, int enable);
/* Accumulated ms per RDM_PH_* phase and launches per phase since the last
 * reset (synchronises the stream). */
rdm_status rdm_get_phase_times(rdm_ctx* ctx, double* ms, int64_t* launches);
rdm_status rdm_reset_phase_times(rdm_ctx* ctx);

/* Debug: route every NN/NT/TN GEMM to the SIMT fp32 kernel (disable != 0)
 * instead of the tcgen05 3xTF32 kernel (0, default).  Process-wide; for
 * cross-checking the two GEMM paths.  Returns 0. */
int rdm_debug_disable_tc(int disable);

#ifdef __cplusplus
}
#endif
#endif /* RDM_H */
