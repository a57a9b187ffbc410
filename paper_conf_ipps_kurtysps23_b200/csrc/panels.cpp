// panels.cpp — partial replication of the adjacency, R_A < P (§III-E,
// PAPER.md L146-167, Fig. 6; the "Comm. (R_A < P)" rows of Tables II/III and
// §IV-A.4).  SURVEY §8(f) NEXT-4.
//
// P GPUs form a grid of P/R_A row panels × R_A column groups, rank
// p = i·R_A + j.  Panel i of A (rows R_i = row_range(N, P/R_A, i), all N
// columns) is held by the R_A ranks of panel group i, so A is stored R_A times
// in total.  Dense SpMM operands are TILES: rank (i, j) holds rows R_i ×
// columns col_range(f, R_A, j).
//  * SpMM (Fig. 6): out_tile(i, j) = A[R_i, :] · In[:, cols_j]; the input
//    column slice In[:, cols_j] is assembled by broadcasting every tile of
//    column group j to the other P/R_A − 1 members — (P/R_A − 1)·N·f elements
//    per SpMM of width f (L152, L216).
//  * Redistribution row ↔ tile happens inside a panel group only: rank p's
//    row slice row_range(N, P, p) lies in its panel (p ∈ [i R_A, (i+1) R_A)),
//    so the panel's N_i × f block is redistributed among R_A ranks —
//    (R_A − 1)/R_A·N·f elements in total (L214).
// With R_A = P there is one row per panel group … i.e. a panel is the whole
// matrix and the scheme is the full-replication algorithm of the rest of the
// library; with R_A = 1 it is CAGNET's 1D algorithm (L152).
#include <algorithm>
#include <cstring>
#include <vector>

#include "internal.h"

namespace rdm {

namespace {
Range panel_rows(int64_t n, int P, int RA, int i) { return row_range(n, P / RA, i); }

struct Grid {
  int P, RA, PI;   // world, column groups (= replicas of A), row panels
  int pi(int p) const { return p / RA; }
  int pj(int p) const { return p % RA; }
};

Grid grid_of(const rdm_ctx* ctx) {
  RDM_CHECK_ARG(ctx->panel_RA > 0, "panels: no row panels (call rdm_set_graph_panels)");
  return Grid{ctx->world, ctx->panel_RA, ctx->world / ctx->panel_RA};
}
}  // namespace

// Host: install the row panels this process needs.
void set_graph_panels(rdm_ctx* ctx, int RA, int64_t n, int64_t nnz, const int64_t* rowptr,
                      const int32_t* col, const float* val, int on_host) {
  const int P = ctx->world;
  RDM_CHECK_ARG(RA >= 1 && RA <= P && P % RA == 0, "set_graph_panels: R_A must divide P");
  RDM_CHECK_ARG(n >= 0 && nnz >= 0 && rowptr && (nnz == 0 || (col && val)), "set_graph_panels: bad args");
  RDM_CHECK_ARG(n < (int64_t)INT32_MAX, "set_graph_panels: N must fit int32 column indices");
  std::vector<int64_t> rp(n + 1);
  RDM_CUDA(cudaMemcpy(rp.data(), rowptr, (n + 1) * sizeof(int64_t),
                      on_host ? cudaMemcpyHostToHost : cudaMemcpyDeviceToHost));
  RDM_CHECK_ARG(rp[0] == 0 && rp[n] == nnz, "set_graph_panels: rowptr must run 0..nnz");
  const int PI = P / RA;
  ctx->panel_RA = 0;
  ctx->panels.clear();
  ctx->panels.resize(PI);
  for (int s = 0; s < ctx->nlocal(); ++s) {
    const int i = ctx->local[s] / RA;
    if (ctx->panels[i]) continue;
    const Range r = panel_rows(n, P, RA, i);
    std::vector<int64_t> prp(r.size() + 1);
    for (int64_t k = 0; k <= r.size(); ++k) prp[k] = rp[r.lo + k] - rp[r.lo];
    const int64_t pnnz = prp[r.size()];
    auto A = std::make_unique<Csr>();
    const int64_t off = rp[r.lo];
    A->n = r.size();
    A->nnz = pnnz;
    A->rowptr.reset(new DevBuf((r.size() + 1) * sizeof(int64_t)));
    A->col.reset(new DevBuf(std::max<int64_t>(pnnz, 1) * sizeof(int32_t)));
    A->val.reset(new DevBuf(std::max<int64_t>(pnnz, 1) * sizeof(float)));
    RDM_CUDA(cudaMemcpy(A->rowptr->ptr, prp.data(), (r.size() + 1) * sizeof(int64_t), cudaMemcpyHostToDevice));
    if (pnnz) {
      const cudaMemcpyKind k = on_host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
      RDM_CUDA(cudaMemcpy(A->col->ptr, col + off, pnnz * sizeof(int32_t), k));
      RDM_CUDA(cudaMemcpy(A->val->ptr, val + off, pnnz * sizeof(float), k));
    }
    A->n_in = n;
    const int bad = validate_csr(ctx, A->rowptr->as<int64_t>(), A->col->as<int32_t>(), r.size(), pnnz);
    // validate_csr checks columns < its n: re-check against N on the host side
    // only when the panel is square-incompatible (columns up to N − 1 are legal)
    RDM_CHECK_ARG((bad & ~1) == 0, "set_graph_panels: invalid rowptr");
    if (bad & 1) {
      std::vector<int32_t> hc(pnnz);
      RDM_CUDA(cudaMemcpy(hc.data(), A->col->ptr, pnnz * sizeof(int32_t), cudaMemcpyDeviceToHost));
      for (int32_t c : hc) RDM_CHECK_ARG(c >= 0 && c < n, "set_graph_panels: column out of range");
    }
    build_bins(ctx, *A, prp.data());
    ctx->panels[i] = std::move(A);
  }
  RDM_CUDA(cudaDeviceSynchronize());
  ctx->panel_RA = RA;
  ctx->panel_n = n;
}

// Tile layout of rank p: rows R_i, columns col_range(f, R_A, j), ld = roundup4(width).
void tile_of(int P, int RA, int64_t n, int64_t f, int p, Range* rows, Range* cols, int64_t* ld) {
  *rows = panel_rows(n, P, RA, p / RA);
  *cols = col_range(f, RA, p % RA);
  *ld = roundup4(cols->size());
}

// Row slices ↔ tiles inside each panel group (all-to-all among R_A ranks).
void redistribute_panels(rdm_ctx* ctx, rdm_layout from, const float* const* src, float* const* dst,
                         int64_t n, int64_t f) {
  const Grid G = grid_of(ctx);
  RDM_CHECK_ARG(n == ctx->panel_n, "redistribute_panels: n differs from the installed graph");
  RDM_CHECK_ARG(G.RA <= BlockTable::kMax, "redistribute_panels: R_A too large");
  const int P = G.P, nl = ctx->nlocal();
  const int64_t ld_row = roundup4(f);
  if ((int)ctx->ws_send.size() < nl) {
    ctx->ws_send.resize(nl);
    ctx->ws_recv.resize(nl);
  }
  std::vector<Xfer> x(nl);
  std::vector<BlockTable> bt(nl);
  int64_t payload = 0, wire = 0;
  for (int s = 0; s < nl; ++s) {
    std::memset(&x[s], 0, sizeof(Xfer));
    const int p = ctx->local[s];
    const int i = G.pi(p), jp = G.pj(p);
    const Range R = panel_rows(n, P, G.RA, i);
    const Range mine = row_range(n, P, p);
    const int64_t rp = mine.size();
    const int64_t ld_p = roundup4(col_range(f, G.RA, jp).size());
    float* stage = ensure_ws(from == RDM_ROW ? ctx->ws_send[s] : ctx->ws_recv[s],
                             (size_t)std::max<int64_t>(rp * ld_row, 1) * sizeof(float));
    int64_t off = 0;
    for (int j = 0; j < G.RA; ++j) {   // member j of my panel group = rank i·R_A + j
      const int q = i * G.RA + j;
      const Range cq = col_range(f, G.RA, j);
      const Range rq = row_range(n, P, q);
      const int64_t ldq = roundup4(cq.size());
      bt[s].col_lo[j] = cq.lo;
      bt[s].width[j] = cq.size();
      bt[s].ld[j] = ldq;
      float* blk = stage + off;
      off += rp * ldq;
      if (from == RDM_ROW) {
        bt[s].dst[j] = (q == p) ? dst[s] + (mine.lo - R.lo) * ld_p : blk;
        x[s].send[q] = blk;
        x[s].send_bytes[q] = (q == p) ? 0 : rp * ldq * sizeof(float);
        x[s].recv[q] = dst[s] + (rq.lo - R.lo) * ld_p;
        x[s].recv_bytes[q] = (q == p) ? 0 : rq.size() * ld_p * sizeof(float);
        if (q != p) payload += rp * cq.size();
      } else {
        bt[s].src[j] = (q == p) ? src[s] + (mine.lo - R.lo) * ld_p : blk;
        x[s].send[q] = src[s] + (rq.lo - R.lo) * ld_p;
        x[s].send_bytes[q] = (q == p) ? 0 : rq.size() * ld_p * sizeof(float);
        x[s].recv[q] = blk;
        x[s].recv_bytes[q] = (q == p) ? 0 : rp * ldq * sizeof(float);
        if (q != p) payload += rq.size() * col_range(f, G.RA, jp).size();
      }
      wire += x[s].send_bytes[q];
    }
  }
  if (from == RDM_ROW) {
    {
      Phase ph(ctx, RDM_PH_PACK);
      for (int s = 0; s < nl; ++s)
        pack_rows(ctx, src[s], ld_row, row_range(n, P, ctx->local[s]).size(), G.RA, bt[s]);
    }
    if (P > 1) exchange(ctx, x);
  } else {
    if (P > 1) exchange(ctx, x);
    Phase ph(ctx, RDM_PH_PACK);
    for (int s = 0; s < nl; ++s)
      unpack_rows(ctx, dst[s], ld_row, row_range(n, P, ctx->local[s]).size(), G.RA, bt[s]);
  }
  ctx->counters.a2a_calls++;
  ctx->counters.a2a_elems_payload += payload;
  ctx->counters.a2a_bytes_wire += wire;
  ctx->counters.a2a_width_units += f;
}

// Fig. 6 SpMM: broadcast the tiles of each column group, then multiply the
// local row panel by the assembled N x w_j column slice.
void spmm_panels(rdm_ctx* ctx, const float* const* in, float* const* out, int64_t f, int epi,
                 const float* bias, const float* const* mask) {
  const Grid G = grid_of(ctx);
  const int P = G.P, nl = ctx->nlocal();
  const int64_t n = ctx->panel_n;
  std::vector<float*> full(nl);
  std::vector<int64_t> ldj(nl);
  size_t per = 0;
  for (int s = 0; s < nl; ++s) {
    ldj[s] = roundup4(col_range(f, G.RA, G.pj(ctx->local[s])).size());
    per = std::max<size_t>(per, (size_t)n * ldj[s]);
  }
  per = (per + 63) / 64 * 64;
  float* ws = ensure_ws(ctx->ws_panel_in, std::max<size_t>(per * nl, 64) * sizeof(float));
  std::vector<Xfer> x(nl);
  int64_t bcast = 0;
  for (int s = 0; s < nl; ++s) {
    std::memset(&x[s], 0, sizeof(Xfer));
    full[s] = ws + per * s;
    const int p = ctx->local[s];
    const int i = G.pi(p), j = G.pj(p);
    const Range R = panel_rows(n, P, G.RA, i);
    // my own tile goes to its place in the assembled slice
    if (R.size() && ldj[s])
      RDM_CUDA(cudaMemcpyAsync(full[s] + R.lo * ldj[s], in[s], R.size() * ldj[s] * sizeof(float),
                               cudaMemcpyDeviceToDevice, ctx->stream));
    for (int i2 = 0; i2 < G.PI; ++i2) {
      if (i2 == i) continue;
      const int q = i2 * G.RA + j;      // same column group
      const Range Rq = panel_rows(n, P, G.RA, i2);
      x[s].send[q] = in[s];
      x[s].send_bytes[q] = R.size() * ldj[s] * sizeof(float);
      x[s].recv[q] = full[s] + Rq.lo * ldj[s];
      x[s].recv_bytes[q] = Rq.size() * ldj[s] * sizeof(float);
      bcast += R.size() * col_range(f, G.RA, j).size();
    }
  }
  if (P > 1 && G.PI > 1) exchange(ctx, x);
  Phase ph(ctx, RDM_PH_SPMM);
  for (int s = 0; s < nl; ++s) {
    const int p = ctx->local[s];
    const Csr& A = *ctx->panels[G.pi(p)];
    const int64_t w = col_range(f, G.RA, G.pj(p)).size();
    spmm(ctx, A, full[s], ldj[s], out[s], ldj[s], w, epi, bias ? bias + col_range(f, G.RA, G.pj(p)).lo : nullptr,
         mask ? mask[s] : nullptr, ldj[s]);
  }
  ctx->counters.spmm_width_units += f;
  ctx->counters.bcast_elems += bcast;
}

// Largest R_A (a divisor of P, at most P) whose replicas fit (L160-167,
// reading R36); 0 if one copy of A does not fit in the aggregate memory.
int max_replication(int P, double mem_bytes, double h_all_bytes, double g_bytes) {
  const double bound = g_bytes > 0 ? P * (mem_bytes - h_all_bytes) / g_bytes : (double)P;
  const int cap = bound >= 1 ? (int)std::min<double>(P, bound) : 0;
  for (int r = cap; r >= 1; --r)
    if (P % r == 0) return r;
  return 0;
}

}  // namespace rdm
