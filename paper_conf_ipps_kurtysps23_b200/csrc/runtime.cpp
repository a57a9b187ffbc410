// runtime.cpp — context, graph residency, transport (NCCL / virtual group),
// redistribution driver and the C ABI entry points of rdm.h (except the GCN
// executor in gcn.cpp and the cost model in plan.cpp).
#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include "internal.h"

namespace rdm {

int validate_csr(rdm_ctx* ctx, const int64_t* rowptr, const int32_t* col, int64_t n, int64_t nnz);
void gemm_simt(rdm_ctx* ctx, int op, const float* X, int64_t ldx, const float* W, int64_t ldw,
               float* C, int64_t ldc, int64_t rows, int64_t k, int64_t m, int epi,
               const float* bias, const float* mask);
bool gemm_tc(rdm_ctx* ctx, int op, const float* X, int64_t ldx, const float* W, int64_t ldw,
             float* C, int64_t ldc, int64_t rows, int64_t k, int64_t m, int epi, const float* bias,
             const float* mask, const Scatter* scat);

#define RDM_NCCL(call)                                                                     \
  do {                                                                                     \
    ncclResult_t r_ = (call);                                                              \
    if (r_ != ncclSuccess)                                                                 \
      throw ::rdm::Error(RDM_ERR_NCCL, std::string(#call) + ": " + ncclGetErrorString(r_)); \
  } while (0)

// ---------------------------------------------------------------- partition
Range row_range(int64_t n, int P, int p) { return {(int64_t)p * n / P, (int64_t)(p + 1) * n / P}; }

Range col_range(int64_t f, int P, int p) {
  const int64_t g = (f + 3) / 4;
  auto lo = [&](int q) -> int64_t { return q >= P ? f : std::min<int64_t>(f, 4 * ((q * g) / P)); };
  return {lo(p), p + 1 < P ? lo(p + 1) : f};
}

// ------------------------------------------------------------------ memory
DevBuf::DevBuf(size_t b) : bytes(b) {
  if (b) {
    cudaError_t e = cudaMalloc(&ptr, b);
    if (e != cudaSuccess) {
      ptr = nullptr;
      (void)cudaGetLastError();
      throw Error(RDM_ERR_OOM, "cudaMalloc(" + std::to_string(b) + " B) failed: " +
                                   cudaGetErrorString(e));
    }
  }
}
DevBuf::~DevBuf() {
  if (ptr) cudaFree(ptr);
}

// Workspace diagnostics, read on every call (tests may set them at any time):
// RDM_WS_LOG=1 logs every regrowth; RDM_WS_HEADROOM = percent of headroom on a
// regrowth (default 25, clamped to 0..400).
static bool ws_log() {
  const char* v = getenv("RDM_WS_LOG");
  return v && atoi(v) > 0;
}
static size_t ws_headroom_pct() {
  const char* v = getenv("RDM_WS_HEADROOM");
  if (!v) return 25;
  const long x = strtol(v, nullptr, 10);
  return (size_t)std::min<long>(400, std::max<long>(0, x));
}

namespace {
std::mutex g_retired_mu;
std::vector<void*> g_retired_dev, g_retired_host;
}  // namespace

void retire(void* dev_ptr, void* host_ptr) {
  std::lock_guard<std::mutex> lk(g_retired_mu);
  if (dev_ptr) g_retired_dev.push_back(dev_ptr);
  if (host_ptr) g_retired_host.push_back(host_ptr);
}

void release_retired() {
  std::vector<void*> d, h;
  {
    std::lock_guard<std::mutex> lk(g_retired_mu);
    d.swap(g_retired_dev);
    h.swap(g_retired_host);
  }
  for (void* p : d) cudaFree(p);       // synchronises the device: only at sync points
  for (void* p : h) cudaFreeHost(p);
}

float* ensure_ws(std::unique_ptr<DevBuf>& b, size_t bytes) {
  if (!b || b->bytes < bytes) {
    // regrowth (sizes that vary per call, e.g. GraphSAINT subgraphs) gets
    // headroom so that it stays rare; the old buffer is retired, not freed
    // (cudaFree would synchronise the device in the middle of a step)
    const size_t want = b ? bytes + bytes * ws_headroom_pct() / 100 : bytes;
    if (b && ws_log()) fprintf(stderr, "[rdm ws] regrow %zu -> %zu\n", b->bytes, want);
    std::unique_ptr<DevBuf> nb(new DevBuf(std::max<size_t>(want, 256)));
    if (b) {
      retire(b->ptr, nullptr);
      b->ptr = nullptr;
    }
    b = std::move(nb);
  }
  return b->as<float>();
}

Pinned::~Pinned() {
  if (p) cudaFreeHost(p);
}

void Pinned::reserve(size_t want) {
  if (want <= bytes) return;
  const size_t nb = want + want / 4;
  if (p && ws_log()) fprintf(stderr, "[rdm ws] pinned regrow %zu -> %zu\n", bytes, nb);
  void* q = nullptr;
  if (cudaMallocHost(&q, nb) != cudaSuccess) {
    (void)cudaGetLastError();
    throw Error(RDM_ERR_OOM, "pinned host buffer of " + std::to_string(nb) + " B");
  }
  if (p) retire(nullptr, p);
  p = q;
  bytes = nb;
}

// ------------------------------------------------------------------- timing
Phase::Phase(rdm_ctx* c, int ph) : ctx(c), prev(c->cur_phase) {
  ctx->cur_phase = ph;
  if (ctx->timing) {
    if (ctx->event_pool.empty()) {
      cudaEvent_t e;
      RDM_CUDA(cudaEventCreate(&e));
      ctx->event_pool.push_back(e);
    }
    a = ctx->event_pool.back();
    ctx->event_pool.pop_back();
    RDM_CUDA(cudaEventRecord(a, ctx->stream));
  }
}
Phase::~Phase() {
  if (ctx->timing && a) {
    cudaEvent_t b;
    if (ctx->event_pool.empty()) {
      if (cudaEventCreate(&b) != cudaSuccess) b = nullptr;
    } else {
      b = ctx->event_pool.back();
      ctx->event_pool.pop_back();
    }
    if (b) {
      cudaEventRecord(b, ctx->stream);
      ctx->events.push_back({ctx->cur_phase, a, b});
    }
  }
  ctx->cur_phase = prev;
}

static void drain_events(rdm_ctx* ctx) {
  if (ctx->events.empty()) return;
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  for (auto& e : ctx->events) {
    // phases may have been recorded on another stream (the GraphSAINT sampler's)
    RDM_CUDA(cudaEventSynchronize(e.b));
    float ms = 0;
    RDM_CUDA(cudaEventElapsedTime(&ms, e.a, e.b));
    ctx->phase_ms[e.phase] += ms;
    ctx->event_pool.push_back(e.a);
    ctx->event_pool.push_back(e.b);
  }
  ctx->events.clear();
}

// --------------------------------------------------------------- transport
void exchange(rdm_ctx* ctx, std::vector<Xfer>& x) {
  const int P = ctx->world;
  Phase ph(ctx, RDM_PH_A2A);
  if (ctx->virtual_group()) {
    for (int p = 0; p < P; ++p)
      for (int q = 0; q < P; ++q) {
        if (q == p) continue;
        const size_t b = x[p].send_bytes[q];
        if (b != x[q].recv_bytes[p])
          throw Error(RDM_ERR_STATE, "virtual exchange: send/recv size mismatch");
        if (b) RDM_CUDA(cudaMemcpyAsync(x[q].recv[p], x[p].send[q], b, cudaMemcpyDeviceToDevice,
                                        ctx->stream));
      }
    return;
  }
  if (P == 1 || ctx->emulated) return;   // emulated rank: no peers, nothing crosses a link
  const int p = ctx->rank;
  RDM_NCCL(ncclGroupStart());
  for (int q = 0; q < P; ++q) {
    if (q == p) continue;
    if (x[0].send_bytes[q])
      RDM_NCCL(ncclSend(x[0].send[q], x[0].send_bytes[q] / 4, ncclFloat, q, ctx->comm, ctx->stream));
    if (x[0].recv_bytes[q])
      RDM_NCCL(ncclRecv(x[0].recv[q], x[0].recv_bytes[q] / 4, ncclFloat, q, ctx->comm, ctx->stream));
  }
  RDM_NCCL(ncclGroupEnd());
}

void allreduce(rdm_ctx* ctx, float* const* bufs, int64_t count) {
  if (ctx->world == 1 || count == 0) return;
  Phase ph(ctx, RDM_PH_ALLREDUCE);
  if (ctx->virtual_group()) {
    std::vector<const float*> parts(bufs, bufs + ctx->nlocal());
    sum_slots(ctx, bufs[0], parts.data(), ctx->nlocal(), count);  // ordered sum, in place on slot 0
    for (int i = 1; i < ctx->nlocal(); ++i)
      RDM_CUDA(cudaMemcpyAsync(bufs[i], bufs[0], count * sizeof(float), cudaMemcpyDeviceToDevice,
                               ctx->stream));
  } else if (!ctx->emulated) {
    RDM_NCCL(ncclAllReduce(bufs[0], bufs[0], count, ncclFloat, ncclSum, ctx->comm, ctx->stream));
  }
  ctx->counters.allreduce_bytes += count * 4;
}

void allreduce_d(rdm_ctx* ctx, double* const* bufs, int64_t count) {
  if (ctx->world == 1 || count == 0) return;
  Phase ph(ctx, RDM_PH_ALLREDUCE);
  if (ctx->virtual_group()) {
    RDM_CHECK_ARG(count == 1, "allreduce_d: virtual group supports scalars");
    std::vector<const double*> parts(bufs, bufs + ctx->nlocal());
    double* tmp = reinterpret_cast<double*>(ensure_ws(ctx->ws_scratch, 4096)) + 256;
    sum_doubles(ctx, tmp, parts.data(), ctx->nlocal());
    for (int i = 0; i < ctx->nlocal(); ++i)
      RDM_CUDA(cudaMemcpyAsync(bufs[i], tmp, sizeof(double), cudaMemcpyDeviceToDevice, ctx->stream));
  } else if (!ctx->emulated) {
    RDM_NCCL(ncclAllReduce(bufs[0], bufs[0], count, ncclDouble, ncclSum, ctx->comm, ctx->stream));
  }
  ctx->counters.allreduce_bytes += count * 8;
}

// ---------------------------------------------------------- redistribution
// RDM_PREC_FAST inside the executor: the same exchange
// with bf16 blocks on the wire (half the bytes of L142's (P−1)/P·N·f).  Both
// sides stage: row→col packs bf16 blocks and the receiver widens its staged
// column slice; col→row narrows the sender's column slice and the receiver
// unpacks bf16 blocks.  Every moved value, and the self block, is rounded
// once to bf16 (the fast variant's 2e-2 gate; the public rdm_redistribute
// stays bit-exact fp32).
static void redistribute_bf16(rdm_ctx* ctx, rdm_layout from, const float* const* src, float* const* dst,
                              int64_t n, int64_t f) {
  const int P = ctx->world;
  const int64_t ld_row = roundup4(f);
  std::vector<Range> rows(P), cols(P);
  std::vector<int64_t> ldc(P);
  for (int q = 0; q < P; ++q) {
    rows[q] = row_range(n, P, q);
    cols[q] = col_range(f, P, q);
    ldc[q] = roundup4(cols[q].size());
  }
  const int nl = ctx->nlocal();
  if ((int)ctx->ws_send.size() < nl) {
    ctx->ws_send.resize(nl);
    ctx->ws_recv.resize(nl);
  }
  std::vector<Xfer> x(nl);
  std::vector<BlockTable> bt(nl);
  std::vector<uint16_t*> rowstage(nl), colstage(nl);
  int64_t payload = 0, wire = 0;
  for (int i = 0; i < nl; ++i) {
    const int p = ctx->local[i];
    const int64_t rp = rows[p].size();
    auto& rs = from == RDM_ROW ? ctx->ws_send[i] : ctx->ws_recv[i];   // row-side staging: P blocks
    auto& cs = from == RDM_ROW ? ctx->ws_recv[i] : ctx->ws_send[i];   // column-side staging: N x ld_p
    rowstage[i] = reinterpret_cast<uint16_t*>(ensure_ws(rs, (size_t)std::max<int64_t>(rp * ld_row, 1) * 2 + 64));
    colstage[i] = reinterpret_cast<uint16_t*>(ensure_ws(cs, (size_t)std::max<int64_t>(n * ldc[p], 1) * 2 + 64));
    int64_t off = 0;
    for (int q = 0; q < P; ++q) {
      bt[i].col_lo[q] = cols[q].lo;
      bt[i].width[q] = cols[q].size();
      bt[i].ld[q] = ldc[q];
      uint16_t* blk = rowstage[i] + off;
      off += rp * ldc[q];
      bt[i].dst[q] = reinterpret_cast<float*>(blk);
      bt[i].src[q] = reinterpret_cast<const float*>(blk);
      uint16_t* cblk = colstage[i] + rows[q].lo * ldc[p];
      if (from == RDM_ROW) {
        x[i].send[q] = blk;
        x[i].send_bytes[q] = (q == p) ? 0 : rp * ldc[q] * 2;
        x[i].recv[q] = cblk;
        x[i].recv_bytes[q] = (q == p) ? 0 : rows[q].size() * ldc[p] * 2;
        if (q != p) payload += rp * cols[q].size();
      } else {
        x[i].send[q] = cblk;
        x[i].send_bytes[q] = (q == p) ? 0 : rows[q].size() * ldc[p] * 2;
        x[i].recv[q] = blk;
        x[i].recv_bytes[q] = (q == p) ? 0 : rp * ldc[q] * 2;
        if (q != p) payload += rows[q].size() * cols[p].size();
      }
      wire += x[i].send_bytes[q];
    }
  }
  if (from == RDM_ROW) {
    {
      Phase ph(ctx, RDM_PH_PACK);
      for (int i = 0; i < nl; ++i) {
        const int p = ctx->local[i];
        pack_rows_bf16(ctx, src[i], ld_row, rows[p].size(), P, p, bt[i], dst[i] + rows[p].lo * ldc[p], ldc[p]);
      }
    }
    exchange(ctx, x);
    Phase ph(ctx, RDM_PH_PACK);
    for (int i = 0; i < nl; ++i) {
      const int p = ctx->local[i];
      widen_cols(ctx, colstage[i], n, ldc[p], rows[p].lo, rows[p].hi, dst[i]);
    }
  } else {
    {
      Phase ph(ctx, RDM_PH_PACK);
      for (int i = 0; i < nl; ++i) {
        const int p = ctx->local[i];
        narrow_cols(ctx, src[i], n, ldc[p], rows[p].lo, rows[p].hi, colstage[i]);
      }
    }
    exchange(ctx, x);
    Phase ph(ctx, RDM_PH_PACK);
    for (int i = 0; i < nl; ++i) {
      const int p = ctx->local[i];
      unpack_rows_bf16(ctx, dst[i], ld_row, rows[p].size(), P, p, bt[i], src[i] + rows[p].lo * ldc[p], ldc[p]);
    }
  }
  ctx->counters.a2a_calls++;
  ctx->counters.a2a_elems_payload += payload;
  ctx->counters.a2a_bytes_wire += wire;
  ctx->counters.a2a_width_units += f;
}

void redistribute(rdm_ctx* ctx, rdm_layout from, const float* const* src, float* const* dst,
                  int64_t n, int64_t f, bool bf16_wire) {
  const int P = ctx->world;
  if (bf16_wire && P > 1) return redistribute_bf16(ctx, from, src, dst, n, f);
  const int64_t ld_row = roundup4(f);
  if (P == 1) {
    if (src[0] != dst[0] && n * ld_row != 0)
      RDM_CUDA(cudaMemcpyAsync(dst[0], src[0], n * ld_row * sizeof(float), cudaMemcpyDeviceToDevice,
                               ctx->stream));
    ctx->counters.a2a_calls++;
    ctx->counters.a2a_width_units += f;
    return;
  }
  RDM_CHECK_ARG(P <= BlockTable::kMax, "world too large");
  std::vector<Range> rows(P), cols(P);
  std::vector<int64_t> ldc(P);
  for (int q = 0; q < P; ++q) {
    rows[q] = row_range(n, P, q);
    cols[q] = col_range(f, P, q);
    ldc[q] = roundup4(cols[q].size());
  }
  const int nl = ctx->nlocal();
  if ((int)ctx->ws_send.size() < nl) {
    ctx->ws_send.resize(nl);
    ctx->ws_recv.resize(nl);
  }
  std::vector<Xfer> x(nl);
  std::vector<BlockTable> bt(nl);
  int64_t payload = 0, wire = 0;
  for (int i = 0; i < nl; ++i) {
    const int p = ctx->local[i];
    const int64_t rp = rows[p].size();
    float* stage = ensure_ws(from == RDM_ROW ? ctx->ws_send[i] : ctx->ws_recv[i],
                             (size_t)std::max<int64_t>(rp * ld_row, 1) * sizeof(float));
    int64_t off = 0;
    for (int q = 0; q < P; ++q) {
      bt[i].col_lo[q] = cols[q].lo;
      bt[i].width[q] = cols[q].size();
      bt[i].ld[q] = ldc[q];
      float* blk = stage + off;
      off += rp * ldc[q];
      if (from == RDM_ROW) {
        // pack: self block straight into my column slice
        bt[i].dst[q] = (q == p) ? dst[i] + rows[p].lo * ldc[p] : blk;
        x[i].send[q] = blk;
        x[i].send_bytes[q] = (q == p) ? 0 : rp * ldc[q] * sizeof(float);
        x[i].recv[q] = dst[i] + rows[q].lo * ldc[p];
        x[i].recv_bytes[q] = (q == p) ? 0 : rows[q].size() * ldc[p] * sizeof(float);
        if (q != p) payload += rp * cols[q].size();
      } else {
        // unpack reads the self block straight from my column slice
        bt[i].src[q] = (q == p) ? src[i] + rows[p].lo * ldc[p] : blk;
        x[i].send[q] = src[i] + rows[q].lo * ldc[p];
        x[i].send_bytes[q] = (q == p) ? 0 : rows[q].size() * ldc[p] * sizeof(float);
        x[i].recv[q] = blk;
        x[i].recv_bytes[q] = (q == p) ? 0 : rp * ldc[q] * sizeof(float);
        if (q != p) payload += rows[q].size() * cols[p].size();
      }
      wire += x[i].send_bytes[q];
    }
  }
  if (from == RDM_ROW) {
    {
      Phase ph(ctx, RDM_PH_PACK);
      for (int i = 0; i < nl; ++i)
        pack_rows(ctx, src[i], ld_row, rows[ctx->local[i]].size(), P, bt[i]);
    }
    exchange(ctx, x);
  } else {
    exchange(ctx, x);
    Phase ph(ctx, RDM_PH_PACK);
    for (int i = 0; i < nl; ++i)
      unpack_rows(ctx, dst[i], ld_row, rows[ctx->local[i]].size(), P, bt[i]);
  }
  ctx->counters.a2a_calls++;
  ctx->counters.a2a_elems_payload += payload;
  ctx->counters.a2a_bytes_wire += wire;
  ctx->counters.a2a_width_units += f;
}

// A redistribution fused into its producer (RDM_TRANSPORT_P2P): the data
// already moved; count the same logical traffic as redistribute() — payload
// elements and the wire bytes the producer stored into peer memory (real
// elements only: no ld padding crosses the link).
void count_fused_redist(rdm_ctx* ctx, rdm_layout from, int64_t n, int64_t f) {
  const int P = ctx->world;
  int64_t payload = 0;
  for (int i = 0; i < ctx->nlocal(); ++i) {
    const int p = ctx->local[i];
    for (int q = 0; q < P; ++q) {
      if (q == p) continue;
      payload += from == RDM_ROW ? row_range(n, P, p).size() * col_range(f, P, q).size()
                                 : row_range(n, P, q).size() * col_range(f, P, p).size();
    }
  }
  ctx->counters.a2a_calls++;
  ctx->counters.a2a_elems_payload += payload;
  ctx->counters.a2a_bytes_wire += payload * (int64_t)sizeof(float);
  ctx->counters.a2a_width_units += f;
}

// Stream-ordered barrier across NCCL ranks (one-word all-reduce): when it
// completes on my stream, every rank's stream has reached the same point.
// Virtual group / P = 1: stream order already is the barrier.
void p2p_barrier(rdm_ctx* ctx) {
  if (ctx->world == 1 || ctx->virtual_group() || ctx->emulated) return;
  Phase ph(ctx, RDM_PH_A2A);
  float* w = ensure_ws(ctx->ws_scratch, 4096);
  RDM_NCCL(ncclAllReduce(w, w, 1, ncclFloat, ncclSum, ctx->comm, ctx->stream));
}

// Peer base addresses of one device allocation per rank (CUDA IPC, handles
// all-gathered over NCCL).  Virtual group: not used (slots share a process).
std::vector<float*> p2p_open(rdm_ctx* ctx, float* mine, std::vector<void*>& opened) {
  if (ctx->emulated) throw Error(RDM_ERR_UNSUPPORTED, "P2P transport on an emulated rank");
  const int P = ctx->world;
  std::vector<float*> out(P, nullptr);
  out[ctx->rank] = mine;
  cudaIpcMemHandle_t h;
  RDM_CUDA(cudaIpcGetMemHandle(&h, mine));
  constexpr size_t hb = sizeof(cudaIpcMemHandle_t);
  uint8_t* d = reinterpret_cast<uint8_t*>(ensure_ws(ctx->ws_scratch, 4096 + P * hb));
  RDM_CUDA(cudaMemcpyAsync(d + 1024, &h, hb, cudaMemcpyHostToDevice, ctx->stream));
  RDM_NCCL(ncclAllGather(d + 1024, d + 1024 + hb, hb, ncclUint8, ctx->comm, ctx->stream));
  std::vector<cudaIpcMemHandle_t> all(P);
  RDM_CUDA(cudaMemcpyAsync(all.data(), d + 1024 + hb, P * hb, cudaMemcpyDeviceToHost, ctx->stream));
  RDM_CUDA(cudaStreamSynchronize(ctx->stream));
  for (int q = 0; q < P; ++q) {
    if (q == ctx->rank) continue;
    void* ptr = nullptr;
    RDM_CUDA(cudaIpcOpenMemHandle(&ptr, all[q], cudaIpcMemLazyEnablePeerAccess));
    opened.push_back(ptr);
    out[q] = static_cast<float*>(ptr);
  }
  return out;
}

// ------------------------------------------------------------------ graph
void upload_csr(rdm_ctx* ctx, Csr& A, int64_t n, int64_t nnz, const int64_t* rowptr,
                       const int32_t* col, const float* val, bool on_host) {
  A.n = n;
  A.nnz = nnz;
  A.rowptr.reset(new DevBuf((n + 1) * sizeof(int64_t)));
  A.col.reset(new DevBuf(std::max<int64_t>(nnz, 1) * sizeof(int32_t)));
  A.val.reset(new DevBuf(std::max<int64_t>(nnz, 1) * sizeof(float)));
  const cudaMemcpyKind k = on_host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  RDM_CUDA(cudaMemcpy(A.rowptr->ptr, rowptr, (n + 1) * sizeof(int64_t), k));
  if (nnz) {
    RDM_CUDA(cudaMemcpy(A.col->ptr, col, nnz * sizeof(int32_t), k));
    RDM_CUDA(cudaMemcpy(A.val->ptr, val, nnz * sizeof(float), k));
  }
  (void)ctx;
}

static void set_graph(rdm_ctx* ctx, int64_t n, int64_t nnz, const int64_t* rowptr, const int32_t* col,
                      const float* val, int symmetric, int on_host) {
  RDM_CHECK_ARG(n >= 0 && nnz >= 0 && rowptr && (nnz == 0 || (col && val)), "set_graph: bad args");
  RDM_CHECK_ARG(n < (int64_t)INT32_MAX, "set_graph: N must fit int32 column indices");
  Graph& g = ctx->graph;
  ctx->has_graph = false;
  g = Graph();
  g.n = n;
  g.nnz = nnz;
  g.symmetric = symmetric != 0;
  upload_csr(ctx, g.A, n, nnz, rowptr, col, val, on_host);
  const int bad = validate_csr(ctx, g.A.rowptr->as<int64_t>(), g.A.col->as<int32_t>(), n, nnz);
  RDM_CHECK_ARG(bad == 0, "set_graph: invalid CSR (flags " + std::to_string(bad) +
                              ": 1 = column out of range, 2 = rowptr decreasing, 4 = rowptr ends)");
  std::vector<int64_t> rp(n + 1);
  RDM_CUDA(cudaMemcpy(rp.data(), g.A.rowptr->ptr, (n + 1) * sizeof(int64_t), cudaMemcpyDeviceToHost));
  build_bins(ctx, g.A, rp.data());
  if (g.symmetric && nnz > 0) {
    std::vector<int32_t> hc(nnz);
    std::vector<float> hv(nnz);
    RDM_CUDA(cudaMemcpy(hc.data(), g.A.col->ptr, nnz * sizeof(int32_t), cudaMemcpyDeviceToHost));
    RDM_CUDA(cudaMemcpy(hv.data(), g.A.val->ptr, nnz * sizeof(float), cudaMemcpyDeviceToHost));
    if (n >= 4096) build_core(ctx, g.A, rp.data(), hc.data(), hv.data());
    // factorisation a_ij = s_i·s_j of every value (s = deg^-1/2, or all ones)
    // for the fast-precision SpMM's value-free row sums
    std::vector<float> sc(n);
    for (int hyp = 0; hyp < 2 && !g.A.fscale; ++hyp) {
      bool ok = true;
      std::vector<double> sd(n);
      for (int64_t i = 0; i < n; ++i)
        sd[i] = hyp == 0 ? (rp[i + 1] > rp[i] ? 1.0 / std::sqrt((double)(rp[i + 1] - rp[i])) : 0.0) : 1.0;
      for (int64_t i = 0; i < n && ok; ++i)
        for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
          const double f = sd[i] * sd[hc[j]];
          if (!(std::fabs((double)hv[j] - f) <= std::ldexp(f, -21))) {
            ok = false;
            break;
          }
        }
      if (!ok) continue;
      for (int64_t i = 0; i < n; ++i) sc[i] = (float)sd[i];
      g.A.fscale.reset(new DevBuf(std::max<int64_t>(n, 1) * sizeof(float)));
      RDM_CUDA(cudaMemcpy(g.A.fscale->ptr, sc.data(), n * sizeof(float), cudaMemcpyHostToDevice));
    }
  }
  if (!g.symmetric) {
    // Aᵀ as CSR: stable counting sort of (col, row) — one-time setup.
    std::vector<int32_t> c(nnz);
    std::vector<float> v(nnz);
    RDM_CUDA(cudaMemcpy(c.data(), g.A.col->ptr, nnz * sizeof(int32_t), cudaMemcpyDeviceToHost));
    RDM_CUDA(cudaMemcpy(v.data(), g.A.val->ptr, nnz * sizeof(float), cudaMemcpyDeviceToHost));
    std::vector<int64_t> trp(n + 1, 0);
    for (int64_t j = 0; j < nnz; ++j) trp[c[j] + 1]++;
    for (int64_t i = 0; i < n; ++i) trp[i + 1] += trp[i];
    std::vector<int32_t> tc(nnz);
    std::vector<float> tv(nnz);
    std::vector<int64_t> pos(trp.begin(), trp.end() - 1);
    for (int64_t i = 0; i < n; ++i)
      for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
        const int64_t d = pos[c[j]]++;
        tc[d] = (int32_t)i;
        tv[d] = v[j];
      }
    upload_csr(ctx, g.AT, n, nnz, trp.data(), tc.data(), tv.data(), true);
    build_bins(ctx, g.AT, trp.data());
    // hub tiles / dense core for both operators (any square CSR; the tiles
    // need a rank-1 value scaling a_ij = r_i c_j, e.g. a row-normalised graph)
    if (n >= 4096 && nnz > 0) {
      build_core(ctx, g.A, rp.data(), c.data(), v.data());
      build_core(ctx, g.AT, trp.data(), tc.data(), tv.data());
    }
  }
  // hot-row panels of the CSRs the SpMM streams (the hub-core residual if any)
  for (Csr* S : {&g.A, &g.AT}) {
    if (!S->col) continue;
    build_hot(ctx, S->core.resid ? *S->core.resid : *S);
  }
  RDM_CUDA(cudaDeviceSynchronize());
  ctx->has_graph = true;
}

}  // namespace rdm

using namespace rdm;

// ----------------------------------------------------------------- C ABI
template <class F>
static rdm_status guarded(rdm_ctx* ctx, F&& fn) {
  if (!ctx) return RDM_ERR_ARG;
  if (ctx->poisoned) {
    ctx->err = "context poisoned by an earlier NCCL/CUDA fault";
    return RDM_ERR_STATE;
  }
  try {
    int dev = -1;
    cudaGetDevice(&dev);
    if (dev != ctx->device) RDM_CUDA(cudaSetDevice(ctx->device));
    fn();
    return RDM_OK;
  } catch (const Error& e) {
    ctx->err = e.what();
    if (e.status == RDM_ERR_NCCL) {
      if (ctx->comm) ncclCommAbort(ctx->comm);
      ctx->comm = nullptr;
      ctx->poisoned = true;
    }
    if (e.status == RDM_ERR_CUDA) {
      cudaError_t sticky = cudaDeviceSynchronize();
      if (sticky != cudaSuccess) ctx->poisoned = true;
    }
    return e.status;
  } catch (const std::exception& e) {
    ctx->err = e.what();
    return RDM_ERR_STATE;
  }
}

rdm_status rdm_guarded_call(rdm_ctx* ctx, void (*fn)(void*), void* arg);

extern "C" {

rdm_status rdm_get_unique_id(void* id) {
  if (!id) return RDM_ERR_ARG;
  ncclUniqueId u;
  if (ncclGetUniqueId(&u) != ncclSuccess) return RDM_ERR_NCCL;
  static_assert(sizeof(u) == RDM_UNIQUE_ID_BYTES, "unique id size");
  memcpy(id, &u, sizeof(u));
  return RDM_OK;
}

rdm_status rdm_init(rdm_ctx** out, int rank, int world, const void* uid, int device, void* stream) {
  if (!out || world < 1 || world > BlockTable::kMax) return RDM_ERR_ARG;
  if (!(rank == RDM_ALL_RANKS || (rank >= 0 && rank < world))) return RDM_ERR_ARG;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    (void)cudaGetLastError();
    return RDM_ERR_CUDA;
  }
  rdm_ctx* ctx = new rdm_ctx();
  if (const char* e = getenv("RDM_P2P")) ctx->transport = atoi(e) ? RDM_TRANSPORT_P2P : RDM_TRANSPORT_NCCL;
  ctx->world = world;
  ctx->rank = (world == 1) ? 0 : rank;
  ctx->device = device;
  ctx->stream = (cudaStream_t)stream;
  if (ctx->rank == RDM_ALL_RANKS)
    for (int p = 0; p < world; ++p) ctx->local.push_back(p);
  else
    ctx->local.push_back(ctx->rank);
  rdm_status st = guarded(ctx, [&] {
    RDM_CUDA(cudaSetDevice(device));
    RDM_CUDA(cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, device));
    if (world > 1 && rank != RDM_ALL_RANKS) {
      RDM_CHECK_ARG(uid != nullptr, "rdm_init: NCCL unique id required for world > 1");
      ncclUniqueId u;
      memcpy(&u, uid, sizeof(u));
      RDM_NCCL(ncclCommInitRank(&ctx->comm, world, u, rank));
    }
  });
  if (st != RDM_OK) {
    delete ctx;
    return st;
  }
  *out = ctx;
  return RDM_OK;
}

rdm_status rdm_init_emulated(rdm_ctx** out, int rank, int world, int device, void* stream) {
  if (!out || world < 2 || world > BlockTable::kMax || rank < 0 || rank >= world) return RDM_ERR_ARG;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    (void)cudaGetLastError();
    return RDM_ERR_CUDA;
  }
  rdm_ctx* ctx = new rdm_ctx();
  ctx->world = world;
  ctx->rank = rank;
  ctx->emulated = true;
  ctx->device = device;
  ctx->stream = (cudaStream_t)stream;
  ctx->local.push_back(rank);
  rdm_status st = guarded(ctx, [&] {
    RDM_CUDA(cudaSetDevice(device));
    RDM_CUDA(cudaDeviceGetAttribute(&ctx->num_sms, cudaDevAttrMultiProcessorCount, device));
  });
  if (st != RDM_OK) {
    delete ctx;
    return st;
  }
  *out = ctx;
  return RDM_OK;
}

int rdm_is_emulated(const rdm_ctx* ctx) { return ctx && ctx->emulated ? 1 : 0; }

rdm_status rdm_comm_info(rdm_ctx* ctx, int* nccl_version, int* comm_ranks, int* comm_rank,
                         int* comm_device) {
  if (!ctx) return RDM_ERR_ARG;
  return guarded(ctx, [&] {
    int v = 0, n = 0, r = -1, d = -1;
    RDM_NCCL(ncclGetVersion(&v));
    if (ctx->comm) {
      RDM_NCCL(ncclCommCount(ctx->comm, &n));
      RDM_NCCL(ncclCommUserRank(ctx->comm, &r));
      RDM_NCCL(ncclCommCuDevice(ctx->comm, &d));
    }
    if (nccl_version) *nccl_version = v;
    if (comm_ranks) *comm_ranks = n;
    if (comm_rank) *comm_rank = r;
    if (comm_device) *comm_device = d;
  });
}

rdm_status rdm_finalize(rdm_ctx* ctx) {
  if (!ctx) return RDM_ERR_ARG;
  cudaSetDevice(ctx->device);
  if (ctx->stream) cudaStreamSynchronize(ctx->stream);
  else cudaDeviceSynchronize();
  for (auto& e : ctx->events) {
    cudaEventDestroy(e.a);
    cudaEventDestroy(e.b);
  }
  for (auto e : ctx->event_pool) cudaEventDestroy(e);
  if (ctx->aux) {
    cudaStreamSynchronize(ctx->aux);
    cudaStreamDestroy(ctx->aux);
    cudaEventDestroy(ctx->aux_fork);
    cudaEventDestroy(ctx->aux_join);
  }
  if (ctx->comm) ncclCommDestroy(ctx->comm);
  delete ctx;
  release_retired();
  return RDM_OK;
}

const char* rdm_last_error(const rdm_ctx* ctx) { return ctx ? ctx->err.c_str() : "null ctx"; }

rdm_status rdm_sync(rdm_ctx* ctx) {
  return guarded(ctx, [&] {
    RDM_CUDA(cudaStreamSynchronize(ctx->stream));
    release_retired();
    if (ctx->comm) {
      ncclResult_t async_err;
      RDM_NCCL(ncclCommGetAsyncError(ctx->comm, &async_err));
      RDM_NCCL(async_err);
    }
  });
}

rdm_status rdm_set_stream(rdm_ctx* ctx, void* stream) {
  if (!ctx) return RDM_ERR_ARG;
  ctx->stream = (cudaStream_t)stream;
  return RDM_OK;
}

rdm_status rdm_set_transport(rdm_ctx* ctx, int transport) {
  if (!ctx || (transport != RDM_TRANSPORT_NCCL && transport != RDM_TRANSPORT_P2P)) return RDM_ERR_ARG;
  if (ctx->emulated && transport == RDM_TRANSPORT_P2P) {
    ctx->err = "rdm_set_transport: an emulated rank has no peer memory";
    return RDM_ERR_UNSUPPORTED;
  }
  ctx->transport = transport;
  return RDM_OK;
}

int rdm_get_transport(const rdm_ctx* ctx) { return ctx ? ctx->transport : -1; }

rdm_status rdm_set_graph_panels(rdm_ctx* ctx, int R_A, int64_t n, int64_t nnz, const int64_t* rowptr,
                                const int32_t* col, const float* vals, int on_host) {
  return guarded(ctx, [&] { set_graph_panels(ctx, R_A, n, nnz, rowptr, col, vals, on_host); });
}

rdm_status rdm_partition_tile(int world, int R_A, int64_t n, int64_t f, int rank, int64_t* row_lo,
                              int64_t* row_hi, int64_t* col_lo, int64_t* col_hi, int64_t* ld) {
  if (world < 1 || R_A < 1 || R_A > world || world % R_A || rank < 0 || rank >= world || n < 0 || f < 0)
    return RDM_ERR_ARG;
  Range r, c;
  int64_t l;
  tile_of(world, R_A, n, f, rank, &r, &c, &l);
  if (row_lo) *row_lo = r.lo;
  if (row_hi) *row_hi = r.hi;
  if (col_lo) *col_lo = c.lo;
  if (col_hi) *col_hi = c.hi;
  if (ld) *ld = l;
  return RDM_OK;
}

rdm_status rdm_redistribute_panels(rdm_ctx* ctx, rdm_layout from, const float* const* src,
                                   float* const* dst, int64_t n, int64_t f) {
  return guarded(ctx, [&] {
    RDM_CHECK_ARG(src && dst && f >= 0 && (from == RDM_ROW || from == RDM_COL), "redistribute_panels: bad args");
    redistribute_panels(ctx, from, src, dst, n, f);
  });
}

rdm_status rdm_spmm_panels(rdm_ctx* ctx, const float* const* in_tiles, float* const* out_tiles,
                           int64_t f, int epilogue, const float* bias, const float* const* mask_tiles) {
  return guarded(ctx, [&] {
    RDM_CHECK_ARG(in_tiles && out_tiles && f >= 0, "spmm_panels: bad args");
    spmm_panels(ctx, in_tiles, out_tiles, f, epilogue, bias, mask_tiles);
  });
}

int rdm_max_replication(int world, double mem_bytes_per_gpu, double h_all_bytes_per_gpu, double graph_bytes) {
  if (world < 1) return -1;
  return max_replication(world, mem_bytes_per_gpu, h_all_bytes_per_gpu, graph_bytes);
}

rdm_status rdm_set_precision(rdm_ctx* ctx, int precision) {
  if (!ctx || (precision != RDM_PREC_FP32 && precision != RDM_PREC_FAST)) return RDM_ERR_ARG;
  ctx->prec = precision;
  return RDM_OK;
}

int rdm_get_precision(const rdm_ctx* ctx) { return ctx ? ctx->prec : -1; }

int rdm_world(const rdm_ctx* ctx) { return ctx ? ctx->world : -1; }
int rdm_num_local(const rdm_ctx* ctx) { return ctx ? ctx->nlocal() : -1; }
int rdm_local_rank(const rdm_ctx* ctx, int slot) {
  return (ctx && slot >= 0 && slot < ctx->nlocal()) ? ctx->local[slot] : -1;
}

rdm_status rdm_partition(int world, rdm_layout layout, int64_t n, int64_t f, int rank, int64_t* lo,
                         int64_t* hi, int64_t* ld) {
  if (world < 1 || rank < 0 || rank >= world || n < 0 || f < 0) return RDM_ERR_ARG;
  Range r = layout == RDM_ROW ? row_range(n, world, rank) : col_range(f, world, rank);
  if (lo) *lo = r.lo;
  if (hi) *hi = r.hi;
  if (ld) *ld = layout == RDM_ROW ? roundup4(f) : roundup4(r.size());
  return RDM_OK;
}

rdm_status rdm_set_graph(rdm_ctx* ctx, int64_t n, int64_t nnz, const int64_t* rowptr,
                         const int32_t* col, const float* val, int symmetric, int on_host) {
  return guarded(ctx, [&] { set_graph(ctx, n, nnz, rowptr, col, val, symmetric, on_host); });
}

rdm_status rdm_get_graph_info(const rdm_ctx* ctx, rdm_graph_info* out) {
  if (!ctx || !out) return RDM_ERR_ARG;
  if (!ctx->has_graph) return RDM_ERR_STATE;
  const Csr& A = ctx->graph.A;
  *out = rdm_graph_info{};
  out->n = A.n;
  out->nnz = A.nnz;
  out->n_light_rows = A.n_light;
  out->n_heavy_rows = A.n_heavy;
  out->n_segments = A.n_seg;
  out->max_degree = A.max_deg;
  out->core_K = A.core.K;
  out->core_nnz = A.core.nnz;
  out->symmetric = ctx->graph.symmetric ? 1 : 0;
  out->tile_ranks = A.core.K2;
  out->n_tiles = A.core.n_tiles;
  out->n_tile_items = A.core.n_items;
  return RDM_OK;
}

rdm_status rdm_spmm(rdm_ctx* ctx, int transpose, const float* in, int64_t ld_in, float* out,
                    int64_t ld_out, int64_t w, int epilogue, const float* bias, const float* mask,
                    int64_t ld_mask) {
  return guarded(ctx, [&] {
    if (!ctx->has_graph) throw Error(RDM_ERR_STATE, "rdm_spmm: no graph (call rdm_set_graph)");
    Phase ph(ctx, RDM_PH_SPMM);
    const Csr& A = transpose ? ctx->graph.fwd() : ctx->graph.bwd();
    spmm(ctx, A, in, ld_in, out, ld_out, w, epilogue, bias, mask, ld_mask);
  });
}

}  // extern "C"

namespace rdm {
void gemm(rdm_ctx* ctx, int op, const float* X, int64_t ldx, const float* W, int64_t ldw, float* C,
          int64_t ldc, int64_t rows, int64_t k, int64_t m, int epi, const float* bias,
          const float* mask, const Scatter* scat) {
  RDM_CHECK_ARG(op >= 0 && op <= 2 && rows >= 0 && k >= 0 && m >= 0, "gemm: bad op/shape");
  RDM_CHECK_ARG(!scat || (op != RDM_GEMM_TN && scat->mode == 1 && scat->P >= 1 &&
                          scat->P <= Scatter::kMax),
                "gemm: bad scatter descriptor");
  RDM_CHECK_ARG(!(epi & RDM_EPI_BIAS) || bias, "gemm: bias pointer missing");
  RDM_CHECK_ARG(!(epi & RDM_EPI_MASK) || mask, "gemm: mask pointer missing");
  RDM_CHECK_ARG(op != RDM_GEMM_TN || epi == 0, "gemm: TN takes no epilogue");
  ctx->counters.gemm_calls++;
  ctx->counters.gemm_flops += 2 * rows * k * m;
  if (rows == 0 || k == 0 || m == 0) {
    if (op == RDM_GEMM_TN && k && m)
      RDM_CUDA(cudaMemset2DAsync(C, ldc * 4, 0, m * 4, k, ctx->stream));
    return;
  }
  if (gemm_tc(ctx, op, X, ldx, W, ldw, C, ldc, rows, k, m, epi, bias, mask, scat)) return;
  gemm_simt(ctx, op, X, ldx, W, ldw, C, ldc, rows, k, m, epi, bias, mask);
  if (scat) scatter_slice(ctx, C, ldc, rows, op == RDM_GEMM_NN ? m : k, *scat);
}
}  // namespace rdm

extern "C" {

rdm_status rdm_gemm(rdm_ctx* ctx, int op, const float* X, int64_t ldx, const float* W, int64_t ldw,
                    float* C, int64_t ldc, int64_t rows, int64_t k, int64_t m, int epilogue,
                    const float* bias, const float* mask) {
  return guarded(ctx, [&] {
    Phase ph(ctx, RDM_PH_GEMM);
    gemm(ctx, op, X, ldx, W, ldw, C, ldc, rows, k, m, epilogue, bias, mask);
  });
}

rdm_status rdm_redistribute(rdm_ctx* ctx, rdm_layout from, const float* const* src,
                            float* const* dst, int64_t n, int64_t f) {
  return guarded(ctx, [&] {
    RDM_CHECK_ARG(src && dst && n >= 0 && f >= 0, "redistribute: bad args");
    redistribute(ctx, from, src, dst, n, f);
  });
}

rdm_status rdm_allreduce_sum(rdm_ctx* ctx, float* const* bufs, int64_t count) {
  return guarded(ctx, [&] {
    RDM_CHECK_ARG(bufs && count >= 0, "allreduce: bad args");
    allreduce(ctx, bufs, count);
  });
}

rdm_status rdm_adam_step(rdm_ctx* ctx, int count, float* const* params, const float* const* grads,
                         float* const* m, float* const* v, const int64_t* sizes, float lr,
                         float beta1, float beta2, float eps, int step) {
  return guarded(ctx, [&] {
    RDM_CHECK_ARG(count >= 0 && step >= 1, "adam: bad args");
    Phase ph(ctx, RDM_PH_ADAM);
    const float bc1 = (float)(1.0 - std::pow((double)beta1, step));
    const float bc2 = (float)(1.0 - std::pow((double)beta2, step));
    for (int i = 0; i < count; ++i)
      adam(ctx, params[i], grads[i], m[i], v[i], sizes[i], lr, beta1, beta2, eps, bc1, bc2);
  });
}

rdm_status rdm_get_counters(const rdm_ctx* ctx, rdm_counters* out) {
  if (!ctx || !out) return RDM_ERR_ARG;
  *out = ctx->counters;
  return RDM_OK;
}

rdm_status rdm_reset_counters(rdm_ctx* ctx) {
  if (!ctx) return RDM_ERR_ARG;
  ctx->counters = rdm_counters{};
  return RDM_OK;
}

rdm_status rdm_set_timing(rdm_ctx* ctx, int enable) {
  if (!ctx) return RDM_ERR_ARG;
  ctx->timing = enable != 0;
  return RDM_OK;
}

rdm_status rdm_get_phase_times(rdm_ctx* ctx, double* ms, int64_t* launches) {
  return guarded(ctx, [&] {
    drain_events(ctx);
    for (int i = 0; i < RDM_PH_COUNT; ++i) {
      if (ms) ms[i] = ctx->phase_ms[i];
      if (launches) launches[i] = ctx->phase_launches[i];
    }
  });
}

rdm_status rdm_reset_phase_times(rdm_ctx* ctx) {
  return guarded(ctx, [&] {
    drain_events(ctx);
    for (int i = 0; i < RDM_PH_COUNT; ++i) {
      ctx->phase_ms[i] = 0;
      ctx->phase_launches[i] = 0;
    }
  });
}

}  // extern "C"

// exported for gcn.cpp
rdm_status rdm_guarded_call(rdm_ctx* ctx, void (*fn)(void*), void* arg) {
  return guarded(ctx, [&] { fn(arg); });
}

extern "C" rdm_status rdm_redist_plan(int world, int rank, rdm_layout from, int64_t n, int64_t f,
                                      int64_t* send_off, int64_t* send_elems, int64_t* recv_off,
                                      int64_t* recv_elems) {
  if (world < 1 || world > BlockTable::kMax || rank < 0 || rank >= world || n < 0 || f < 0)
    return RDM_ERR_ARG;
  const int P = world, p = rank;
  std::vector<Range> rows(P), cols(P);
  std::vector<int64_t> ldc(P);
  for (int q = 0; q < P; ++q) {
    rows[q] = row_range(n, P, q);
    cols[q] = col_range(f, P, q);
    ldc[q] = roundup4(cols[q].size());
  }
  const int64_t rp = rows[p].size();
  int64_t off = 0;
  for (int q = 0; q < P; ++q) {
    const int64_t stage_off = off;
    off += rp * ldc[q];
    int64_t so, se, ro, re;
    if (from == RDM_ROW) {  // send from staging (packed blocks), recv into my column slice
      so = stage_off; se = rp * ldc[q];
      ro = rows[q].lo * ldc[p]; re = rows[q].size() * ldc[p];
    } else {                // send from my column slice, recv into staging
      so = rows[q].lo * ldc[p]; se = rows[q].size() * ldc[p];
      ro = stage_off; re = rp * ldc[q];
    }
    if (q == p) { se = 0; re = 0; }
    if (send_off) send_off[q] = so;
    if (send_elems) send_elems[q] = se;
    if (recv_off) recv_off[q] = ro;
    if (recv_elems) recv_elems[q] = re;
  }
  return RDM_OK;
}
