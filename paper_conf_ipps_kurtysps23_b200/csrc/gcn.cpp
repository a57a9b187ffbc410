// gcn.cpp — planner + executor of the per-layer GNN-RDM sequence.
//
// PAPER.md §III (L85-167) and §IV (L175-224):
//  * forward layer l, SpMM first (S):  T = Aᵀ H^{l-1} on column slices,
//    redistribute T col→row (kept as the memo T_l, Fig. 4 "T_d saved",
//    L134), Z^l = T W^l on row slices;
//  * forward layer l, GEMM first (D): T = H^{l-1} W^l on row slices,
//    redistribute row→col, Z^l = Aᵀ T on column slices;
//  * H^l = ReLU(Z^l) fused into the producing kernel's epilogue;
//  * the loss needs Z^L row-sliced (L206);
//  * backward layer l, S:  U = A G^l (col), U col→row, Y^l = H^{l-1}ᵀ U,
//    G^{l-1} = U W^{lᵀ} ⊙ σ'(Z^{l-1});  D: V = G^l W^{lᵀ} (row), V row→col,
//    G^{l-1} = (A V) ⊙ σ'(Z^{l-1}), Y^l = T_lᵀ G^l (memo, L120) — or, without
//    the memo, one extra SpMM of width min(f_{l-1}, f_l) (L208, Table III);
//  * every operand is redistributed only when it is not resident in the
//    layout its consumer needs (L210), exactly as the cost model charges.
// The Hadamard σ'(Z^{l-1}) = 1[H^{l-1} > 0] is applied wherever H^{l-1} is
// resident in G^{l-1}'s layout (it commutes with redistribution, reading
// R15); only configurations 6 and 9 (L = 2) must move H^{l-1} for it, which
// the plan reports as hidden communication.
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <map>
#include <set>
#include <sstream>

#include "internal.h"

rdm_status rdm_guarded_call(rdm_ctx* ctx, void (*fn)(void*), void* arg);

namespace rdm {
namespace {

enum Kind { K_H = 0, K_Z, K_T, K_G, K_U, K_V, K_X };
const char* kKindName[] = {"H", "Z", "T", "G", "U", "V", "X"};
struct Key {
  int kind = 0, layer = 0;
  int id() const { return kind * 64 + layer; }
};
enum Op { S_SPMM = 0, S_GEMM, S_TN, S_REDIST, S_MASK, S_LOSS, S_COLSUM };

struct Step {
  int op = 0;
  int trans = 0, gop = 0, epi = 0, wl = 0;
  Key in, in2, out, mask;
  int lin = 0, lin2 = 0, lout = 0, lmask = 0;
  int64_t width = 0;
  bool hidden = false;
  int fuse = 0;   // RDM_TRANSPORT_P2P: 1 = producer also scatters (next step), 2 = redist done by producer
  int bl = 0;     // RDM_GCN_BIAS: layer whose bias b^bl this step adds (0 = none) / sums (S_COLSUM)
};

struct Planner {
  int L = 0, P = 1;
  std::vector<int64_t> f;
  rdm_config cfg{};
  bool igrad = true;
  bool bias = false;   // RDM_GCN_BIAS (reading R8): Z^l = Â H W + 1 b^lᵀ, db^l = 1ᵀ G^l
  std::set<std::pair<int, int>> res, masked;
  std::map<int, int64_t> width;
  std::set<int> pending;
  std::vector<bool> memo;
  std::vector<Step>* cur = nullptr;

  int lay(int l) const { return P == 1 ? 0 : l; }
  bool has(Key k, int l) const {
    return res.count({k.id(), lay(l)}) || (P == 1 && res.count({k.id(), 1}));
  }
  void produce(Key k, int l, int64_t w) {
    res.insert({k.id(), lay(l)});
    width[k.id()] = w;
  }
  void need(Key k, int l, bool hidden) {
    if (has(k, l)) return;
    const int other = 1 - l;
    if (!has(k, other)) throw Error(RDM_ERR_STATE, "planner: operand never produced");
    Step s;
    s.op = S_REDIST;
    s.in = k;
    s.lin = other;
    s.out = k;
    s.lout = l;
    s.width = width[k.id()];
    s.hidden = hidden;
    cur->push_back(s);
    res.insert({k.id(), lay(l)});
    if (masked.count({k.id(), lay(other)})) masked.insert({k.id(), lay(l)});
  }
  void needG(int l, int ly) {
    Key g{K_G, l};
    need(g, ly, false);
    if (l < L && pending.count(g.id()) && !masked.count({g.id(), lay(ly)})) {
      Key h{K_H, l};
      if (!has(h, ly)) need(h, ly, true);
      Step s;
      s.op = S_MASK;
      s.out = g;
      s.lout = ly;
      s.mask = h;
      s.lmask = ly;
      s.width = f[l];
      cur->push_back(s);
      masked.insert({g.id(), lay(ly)});
    }
  }
  void spmm(int trans, Key in, Key out, int64_t w, int epi = 0, Key mask = Key{}) {
    Step s;
    s.op = S_SPMM;
    s.trans = trans;
    s.in = in;
    s.lin = RDM_COL;
    s.out = out;
    s.lout = RDM_COL;
    s.width = w;
    s.epi = epi;
    s.mask = mask;
    s.lmask = RDM_COL;
    cur->push_back(s);
    produce(out, RDM_COL, w);
    if (epi & RDM_EPI_MASK) masked.insert({out.id(), lay(RDM_COL)});
  }
  void gemm(int gop, Key in, int wl, Key out, int64_t w, int epi = 0, Key mask = Key{}) {
    Step s;
    s.op = S_GEMM;
    s.gop = gop;
    s.in = in;
    s.lin = RDM_ROW;
    s.wl = wl;
    s.out = out;
    s.lout = RDM_ROW;
    s.epi = epi;
    s.mask = mask;
    s.lmask = RDM_ROW;
    s.width = w;
    cur->push_back(s);
    produce(out, RDM_ROW, w);
    if (epi & RDM_EPI_MASK) masked.insert({out.id(), lay(RDM_ROW)});
  }
  void colsum(Key gk, int ly, int l) {   // db^l = 1ᵀ G^l from its resident (masked) layout
    Step s;
    s.op = S_COLSUM;
    s.in = gk;
    s.lin = ly;
    s.bl = l;
    s.width = f[l];
    cur->push_back(s);
  }
  void tn(Key x, Key u, int wl) {
    Step s;
    s.op = S_TN;
    s.in = x;
    s.lin = RDM_ROW;
    s.in2 = u;
    s.lin2 = RDM_ROW;
    s.wl = wl;
    cur->push_back(s);
  }

  void plan(std::vector<Step>& fwd, std::vector<Step>& bwd) {
    memo.assign(L + 1, false);
    produce({K_H, 0}, RDM_ROW, f[0]);
    produce({K_H, 0}, RDM_COL, f[0]);
    cur = &fwd;
    for (int l = 1; l <= L; ++l) {
      Key hin{K_H, l - 1}, hout = l < L ? Key{K_H, l} : Key{K_Z, 0}, t{K_T, l};
      const int epi = l < L ? RDM_EPI_RELU : 0;
      const int be = bias ? RDM_EPI_BIAS : 0;   // bias before ReLU, after both products (R8)
      if (!cfg.fwd_D[l - 1]) {
        need(hin, RDM_COL, false);
        spmm(1, hin, t, f[l - 1]);
        need(t, RDM_ROW, false);
        gemm(RDM_GEMM_NN, t, l, hout, f[l], epi | be);
        cur->back().bl = bias ? l : 0;
        memo[l] = true;
      } else {
        need(hin, RDM_ROW, false);
        gemm(RDM_GEMM_NN, hin, l, t, f[l]);
        need(t, RDM_COL, false);
        spmm(1, t, hout, f[l], epi | be);
        cur->back().bl = bias ? l : 0;
      }
    }
    need({K_Z, 0}, RDM_ROW, false);
    {
      Step s;
      s.op = S_LOSS;
      s.in = {K_Z, 0};
      s.lin = RDM_ROW;
      s.out = {K_G, L};
      s.lout = RDM_ROW;
      s.width = f[L];
      fwd.push_back(s);
      produce({K_G, L}, RDM_ROW, f[L]);
    }
    cur = &bwd;
    for (int l = L; l >= 1; --l) {
      Key g{K_G, l}, gout{K_G, l - 1}, hprev{K_H, l - 1}, t{K_T, l};
      const bool out = l > 1 || igrad;
      if (!cfg.bwd_D[l - 1]) {
        needG(l, RDM_COL);
        if (bias) colsum(g, RDM_COL, l);
        Key u{K_U, l};
        spmm(0, g, u, f[l]);
        need(u, RDM_ROW, false);
        if (has(hprev, RDM_ROW)) {
          tn(hprev, u, l);
        } else if (memo[l] && has(g, RDM_ROW) && (l == L || masked.count({g.id(), lay(RDM_ROW)}))) {
          tn(t, g, l);
        } else {
          need(hprev, RDM_ROW, true);
          tn(hprev, u, l);
        }
        if (out) {
          int epi = 0;
          if (l > 1) {
            if (has(hprev, RDM_ROW)) epi = RDM_EPI_MASK;
            else pending.insert(gout.id());
          }
          gemm(RDM_GEMM_NT, u, l, gout, f[l - 1], epi, hprev);
        }
      } else {
        needG(l, RDM_ROW);
        if (bias) colsum(g, RDM_ROW, l);
        Key v{K_V, l};
        gemm(RDM_GEMM_NT, g, l, v, f[l - 1]);
        if (memo[l]) tn(t, g, l);
        if (out) {
          need(v, RDM_COL, false);
          int epi = 0;
          if (l > 1) {
            if (has(hprev, RDM_COL)) epi = RDM_EPI_MASK;
            else pending.insert(gout.id());
          }
          spmm(0, v, gout, f[l - 1], epi, hprev);
        }
        if (!memo[l]) {
          Key x{K_X, l};
          if (f[l - 1] < f[l]) {
            need(hprev, RDM_COL, false);
            spmm(1, hprev, x, f[l - 1]);
            need(x, RDM_ROW, false);
            tn(x, g, l);
          } else {
            needG(l, RDM_COL);
            spmm(0, g, x, f[l]);
            need(x, RDM_ROW, false);
            need(hprev, RDM_ROW, false);
            tn(hprev, x, l);
          }
        }
      }
    }
  }
};

struct Buf {
  float* p = nullptr;
  int64_t rows = 0, cols = 0, ld = 0;
  bool valid_end = true;   // contents still this tensor's after an epoch (RDM_GCN_LOW_MEMORY)
};

// ------------------------------------------------------ workspace planning
// Every (tensor, layout) the plan touches gets a buffer.  Its shape on rank p:
// a row slice (rows of p x ld(f)), a column slice (N x ld(w_p)) or, at
// R_A < P, a tile.  Its lifetime is the step interval [first, last] over the
// epoch's sequence (forward steps, then backward steps; kEnd = the end of the
// epoch).  H^0 row (the input) lives throughout; the operands of the
// weight-gradient GEMMs run on a side stream joined at the end of the
// backward pass, so they live to kEnd; a redistribution's destination may be
// written by its producer one step earlier (fused P2P transport).  H^0's
// column slices, when read, are an input like its row slice: pinned.
// RDM_GCN_LOW_MEMORY: buffers of the same shape whose lifetimes do not
// overlap share one allocation (first-fit, largest first) — same shape, so the
// zero ld-padding every producer keeps stays zero.
constexpr int kEnd = 1 << 20;

struct ShapeCtx {
  int P = 1, p = 0, RA = 0;
  int64_t n_cap = 0;
  bool saint = false;
};

Buf shape_of(const ShapeCtx& sc, int lay, int64_t width) {
  Buf b;
  if (lay == RDM_ROW) {
    b.rows = sc.saint ? ceil_div(sc.n_cap, sc.P) : row_range(sc.n_cap, sc.P, sc.p).size();
    b.cols = width;
    b.ld = roundup4(width);
  } else if (sc.RA) {   // tile: panel rows x column slice over the R_A column groups
    Range r, c;
    tile_of(sc.P, sc.RA, sc.n_cap, width, sc.p, &r, &c, &b.ld);
    b.rows = r.size();
    b.cols = c.size();
  } else {
    b.rows = sc.n_cap;
    b.cols = col_range(width, sc.P, sc.p).size();
    b.ld = roundup4(b.cols);
  }
  return b;
}

struct BufPlan {
  std::pair<int, int> key;   // (tensor id, normalised layout)
  int64_t width = 0;
  int first = kEnd, last = -1;
  Buf shape;
  int slab = -1;
};
struct SlabPlan {
  size_t bytes = 0;
  std::vector<int> members;   // indices into the BufPlan list
};

// Lifetimes of every buffer of the plan (layouts normalised: P = 1 has one).
std::vector<BufPlan> buffer_lifetimes(const Planner& pl, const std::vector<Step>& fwd,
                                      const std::vector<Step>& bwd) {
  std::map<std::pair<int, int>, BufPlan> m;
  auto lay = [&](int l) { return pl.P == 1 ? 0 : l; };
  auto use = [&](Key k, int l, int first, int last) {
    auto key = std::make_pair(k.id(), lay(l));
    BufPlan& b = m[key];
    b.key = key;
    b.width = pl.width.at(k.id());
    b.first = std::min(b.first, first);
    b.last = std::max(b.last, last);
  };
  use({K_H, 0}, RDM_ROW, -1, kEnd);   // the input, set before the epoch
  int t = 0;
  for (auto* v : {&fwd, &bwd})
    for (const Step& s : *v) {
      switch (s.op) {
        case S_SPMM:
        case S_GEMM:
          use(s.in, s.lin, t, t);
          use(s.out, s.lout, t, t);
          if (s.epi & RDM_EPI_MASK) use(s.mask, s.lmask, t, t);
          break;
        case S_TN:
          use(s.in, s.lin, t, kEnd);
          use(s.in2, s.lin2, t, kEnd);
          break;
        case S_REDIST:
          use(s.in, s.lin, t, t);
          use(s.out, s.lout, std::max(0, t - 1), t);
          break;
        case S_MASK:
          use(s.out, s.lout, t, t);
          use(s.mask, s.lmask, t, t);
          break;
        case S_LOSS:
          use(s.in, s.lin, t, t);
          use(s.out, s.lout, t, t);
          break;
        case S_COLSUM:
          use(s.in, s.lin, t, t);
          break;
      }
      ++t;
    }
  // H^0's column slices (when the plan reads them) are an input too: written by
  // set_input before the epoch and read again by the next epoch
  auto h0c = m.find(std::make_pair(Key{K_H, 0}.id(), lay(RDM_COL)));
  if (h0c != m.end()) {
    h0c->second.first = -1;
    h0c->second.last = kEnd;
  }
  std::vector<BufPlan> out;
  for (auto& kv : m) out.push_back(kv.second);
  return out;
}

// Shapes + slab assignment for rank sc.p; returns the slabs, fills b.slab.
std::vector<SlabPlan> plan_slabs(std::vector<BufPlan>& bufs, const ShapeCtx& sc, bool low_memory) {
  for (auto& b : bufs) b.shape = shape_of(sc, b.key.second, b.width);
  auto bytes_of = [](const Buf& s) { return (size_t)std::max<int64_t>(1, s.rows * s.ld) * sizeof(float); };
  std::vector<int> order(bufs.size());
  for (size_t i = 0; i < bufs.size(); ++i) order[i] = (int)i;
  std::stable_sort(order.begin(), order.end(), [&](int a, int b) {
    const size_t ba = bytes_of(bufs[a].shape), bb = bytes_of(bufs[b].shape);
    return ba != bb ? ba > bb : bufs[a].first < bufs[b].first;
  });
  std::vector<SlabPlan> slabs;
  for (int i : order) {
    BufPlan& b = bufs[i];
    int pick = -1;
    if (low_memory) {
      for (size_t k = 0; k < slabs.size() && pick < 0; ++k) {
        const BufPlan& r = bufs[slabs[k].members[0]];
        if (r.shape.rows != b.shape.rows || r.shape.cols != b.shape.cols || r.shape.ld != b.shape.ld) continue;
        bool free = true;
        for (int j : slabs[k].members)
          if (!(bufs[j].last < b.first || b.last < bufs[j].first)) free = false;
        if (free) pick = (int)k;
      }
    }
    if (pick < 0) {
      slabs.push_back({bytes_of(b.shape), {}});
      pick = (int)slabs.size() - 1;
    }
    slabs[pick].members.push_back(i);
    b.slab = pick;
  }
  return slabs;
}

}  // namespace
}  // namespace rdm

using namespace rdm;

struct rdm_gcn {
  rdm_ctx* ctx = nullptr;
  int L = 0, flags = 0;
  std::vector<int64_t> f;
  rdm_config cfg{};
  std::vector<Step> fwd, bwd;
  Planner pl;
  std::vector<std::unique_ptr<DevBuf>> mem;
  // per slot: (key id, layout) → buffer
  std::vector<std::map<std::pair<int, int>, Buf>> bufs;
  std::vector<std::vector<float*>> dwp;     // per slot per layer partial Y (virtual group)
  std::vector<std::vector<float*>> dbp;     // RDM_GCN_BIAS: per slot per layer partial db (virtual group)
  const float* const* bcur = nullptr;       // RDM_GCN_BIAS: the forward pass's b^l (device, f_l floats)
  std::vector<int32_t*> labels;
  std::vector<uint8_t*> mask;
  std::vector<double*> scal;                // per slot: [0] n_train, [1] loss partial
  bool input_set = false;
  // double-buffered host input (see stage_host_input)
  cudaStream_t cs = nullptr;
  cudaEvent_t ev_ready = nullptr, ev_free = nullptr;
  std::vector<float*> st_h0;
  std::vector<int32_t*> st_lab;
  std::vector<uint8_t*> st_mask;
  bool staged = false;
  int64_t ws_bytes = 0;
  rdm_gcn_info info{};
  // fused redistribution (RDM_TRANSPORT_P2P): destination base per rank of
  // every fused (tensor, layout), and the IPC mappings to close at destroy
  bool p2p = false;
  std::map<std::pair<int, int>, std::vector<float*>> peers;
  std::vector<void*> ipc_opened;
  // the graph this instance runs on: the ctx's full graph, or a GraphSAINT
  // sampler's current subgraph (buffers sized for n_cap vertices, row counts
  // refreshed whenever the sampler's version changes)
  const rdm::Graph* graph = nullptr;
  rdm_saint* saint = nullptr;
  int sbuf = 0;           // sampler buffer this instance trains on
  int64_t n_cap = 0;
  // R_A < P (RDM_GCN_PANELS, §III-E): column-layout tensors are tiles of the
  // P/R_A x R_A grid, SpMMs broadcast inside column groups, redistributions
  // stay inside panel groups (panels.cpp).  0 = full replication.
  int RA = 0;
  // weight-gradient GEMMs (S_TN) run on a side stream: they overlap the rest
  // of the backward pass and are joined before the gradient reduction
  cudaStream_t side = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  bool side_pending = false;
  std::unique_ptr<rdm::DevBuf> ws_side;   // split-K partials of the side-stream TN
  int64_t gver = -1;
  // (tensor, layout) whose current contents arrived over the bf16 wire (fast
  // variant): an SpMM reading them uses them as the bf16 values they are
  // (no second rounding of s_j·x_j, rdm_ctx::spmm_in_bf16)
  std::set<std::pair<int, int>> wire_bf16;
  // ReLU sign bits (1/32 of the fp32 Hadamard operand): a row-layout H^l that a
  // GEMM NN produces with ReLU and a later GEMM reads as its mask; per slot
  // one u32 per 32 columns, `mb_valid` once the producer wrote them this epoch
  std::map<std::pair<int, int>, std::vector<uint32_t*>> mbits;
  std::map<std::pair<int, int>, int64_t> mbits_ld;
  std::set<std::pair<int, int>> mb_valid;
};

namespace rdm {
namespace {

int norm_lay(const rdm_gcn* g, int l) { return g->ctx->world == 1 ? 0 : l; }

int64_t gn(const rdm_gcn* g) { return g->RA ? g->ctx->panel_n : g->graph->n; }

// rows a row slice of rank p is allocated for: its share of n_cap, or, for a
// sampler's instance (any n <= n_cap), the largest share ceil(n_cap / P)
int64_t cap_rows(const rdm_gcn* g, int p) {
  const int P = g->ctx->world;
  if (g->saint) return ceil_div(g->n_cap, P);
  return row_range(g->n_cap, P, p).size();
}

// A sampler's instance: after a new subgraph, every buffer's row count
// follows the new vertex count (capacity and leading dims are unchanged).
void sync_graph(rdm_gcn* g) {
  if (!g->saint || g->gver == g->saint->version) return;
  if (g->saint->iteration < 0) throw Error(RDM_ERR_STATE, "GraphSAINT: call rdm_saint_sample first");
  rdm_ctx* ctx = g->ctx;
  // switch to the latest subgraph buffer once its build has finished
  g->graph = &g->saint->graph();
  g->sbuf = g->saint->cur;
  RDM_CUDA(cudaStreamWaitEvent(ctx->stream, g->saint->ev_done[g->sbuf], 0));
  const int64_t n = gn(g);
  for (int s = 0; s < ctx->nlocal(); ++s)
    for (auto& kv : g->bufs[s])
      kv.second.rows = kv.first.second == RDM_ROW ? row_range(n, ctx->world, ctx->local[s]).size() : n;
  g->gver = g->saint->version;
  g->input_set = false;
}

Buf& buf(rdm_gcn* g, int slot, Key k, int l) {
  auto it = g->bufs[slot].find({k.id(), norm_lay(g, l)});
  if (it == g->bufs[slot].end())
    throw Error(RDM_ERR_STATE, std::string("executor: missing buffer ") + kKindName[k.kind] +
                                   std::to_string(k.layer));
  return it->second;
}

void plan_info(const Planner& pl, const std::vector<Step>& fwd, const std::vector<Step>& bwd,
               int64_t n, rdm_gcn_info* out, int RA = 0) {
  rdm_gcn_info in{};
  const int P = pl.P;
  model_costs(pl.L, pl.f.data(), pl.igrad ? 1 : 0, pl.cfg, &in.model_comm_units,
              &in.model_sparse_units);
  auto tot_elems = [&](int64_t w) {
    int64_t t = 0;
    if (P == 1) return t;
    for (int p = 0; p < P; ++p)
      for (int q = 0; q < P; ++q)
        if (p != q && (!RA || p / RA == q / RA))   // R_A < P: inside the panel group only
          t += row_range(n, P, p).size() * (RA ? col_range(w, RA, q % RA) : col_range(w, P, q)).size();
    return t;
  };
  for (auto* v : {&fwd, &bwd})
    for (auto& s : *v) {
      if (s.op == S_REDIST) {
        in.plan_comm_units += s.width;
        if (s.hidden) in.plan_hidden_comm_units += s.width;
        in.a2a_elems += tot_elems(s.width);
      }
      if (s.op == S_SPMM) in.plan_sparse_units += s.width;
    }
  in.n_fwd_steps = (int)fwd.size();
  in.n_bwd_steps = (int)bwd.size();
  *out = in;
}

std::string describe_steps(const std::vector<Step>& fwd, const std::vector<Step>& bwd);

// Fused redistribution (§III-D's all-to-all folded into the producing kernel;
// SURVEY §8(e)): a REDIST whose source the step right before it produced, in
// the producer's own layout (GEMM → row slice → column slices; SpMM → column
// slice → row slices), is replaced by the producer storing each element into
// its owner's destination slice as well.
void setup_fusion(rdm_gcn* g) {
  rdm_ctx* ctx = g->ctx;
  g->p2p = true;
  for (auto* v : {&g->fwd, &g->bwd}) {
    auto& st = *v;
    for (size_t i = 0; i + 1 < st.size(); ++i) {
      Step& a = st[i];
      Step& r = st[i + 1];
      if (r.op != S_REDIST || r.in.id() != a.out.id() || r.lin != a.lout) continue;
      if (!((a.op == S_GEMM && a.lout == RDM_ROW) || (a.op == S_SPMM && a.lout == RDM_COL))) continue;
      a.fuse = 1;
      r.fuse = 2;
      const auto key = std::make_pair(r.out.id(), norm_lay(g, r.lout));
      if (g->peers.count(key)) continue;
      std::vector<float*> ptr(ctx->world, nullptr);
      if (ctx->virtual_group()) {
        for (int q = 0; q < ctx->world; ++q) ptr[q] = buf(g, q, r.out, r.lout).p;
      } else {
        ptr = p2p_open(ctx, buf(g, 0, r.out, r.lout).p, g->ipc_opened);
      }
      g->peers[key] = ptr;
    }
  }
}

// Scatter descriptor of fused producer step `s` for local slot i.
Scatter make_scatter(rdm_gcn* g, const Step& s, int i) {
  rdm_ctx* ctx = g->ctx;
  const int P = ctx->world;
  const int p = ctx->local[i];
  const int64_t n = gn(g), w = s.width;
  const int dl = s.lout == RDM_ROW ? RDM_COL : RDM_ROW;
  const std::vector<float*>& ptr = g->peers.at({s.out.id(), norm_lay(g, dl)});
  Scatter sc;
  sc.P = P;
  if (s.op == S_GEMM) {   // row slice → column slices
    sc.mode = 1;
    for (int q = 0; q < P; ++q) {
      const Range c = col_range(w, P, q);
      sc.lo[q] = c.lo;
      sc.ld[q] = roundup4(c.size());
      sc.ptr[q] = ptr[q];
    }
    sc.lo[P] = w;
    sc.my_off = row_range(n, P, p).lo;
  } else {                // column slice → row slices
    sc.mode = 2;
    for (int q = 0; q < P; ++q) {
      sc.lo[q] = row_range(n, P, q).lo;
      sc.ld[q] = roundup4(w);
      sc.ptr[q] = ptr[q];
    }
    sc.lo[P] = n;
    const Range c = col_range(w, P, p);
    sc.my_off = c.lo;
    sc.my_w = c.size();
  }
  return sc;
}

void create(rdm_gcn* g) {
  rdm_ctx* ctx = g->ctx;
  Planner& pl = g->pl;
  pl.L = g->L;
  pl.P = ctx->world;
  pl.f = g->f;
  pl.cfg = g->cfg;
  pl.igrad = (g->flags & RDM_GCN_INPUT_GRAD) != 0;
  pl.bias = (g->flags & RDM_GCN_BIAS) != 0;
  pl.plan(g->fwd, g->bwd);
  g->bufs.assign(ctx->nlocal(), {});
  const bool low_memory = (g->flags & RDM_GCN_LOW_MEMORY) != 0;
  for (int s = 0; s < ctx->nlocal(); ++s) {
    ShapeCtx sc;
    sc.P = ctx->world;
    sc.p = ctx->local[s];
    sc.RA = g->RA;
    sc.n_cap = g->n_cap;
    sc.saint = g->saint != nullptr;
    std::vector<BufPlan> bp = buffer_lifetimes(pl, g->fwd, g->bwd);
    std::vector<SlabPlan> slabs = plan_slabs(bp, sc, low_memory);
    std::vector<float*> base(slabs.size());
    for (size_t k = 0; k < slabs.size(); ++k) {
      g->mem.emplace_back(new DevBuf(slabs[k].bytes));
      RDM_CUDA(cudaMemset(g->mem.back()->ptr, 0, slabs[k].bytes));
      base[k] = g->mem.back()->as<float>();
      g->ws_bytes += (int64_t)slabs[k].bytes;
    }
    for (const BufPlan& b : bp) {
      Buf x = b.shape;
      x.p = base[b.slab];
      for (int j : slabs[b.slab].members)
        if (bp[j].first > b.first) x.valid_end = false;   // a later tensor reuses this memory
      g->bufs[s][b.key] = x;
    }
  }
  // ReLU sign bits for GEMM → GEMM Hadamards in the row layout (RDM_MASK_BITS=0: off)
  if (!g->RA && !(getenv("RDM_MASK_BITS") && !atoi(getenv("RDM_MASK_BITS")))) {
    std::set<std::pair<int, int>> relu_rows;
    for (auto* v : {&g->fwd, &g->bwd})
      for (const Step& st : *v)
        if (st.op == S_GEMM && (st.epi & RDM_EPI_RELU) && st.lout == RDM_ROW)
          relu_rows.insert({st.out.id(), norm_lay(g, st.lout)});
    for (auto* v : {&g->fwd, &g->bwd})
      for (const Step& st : *v) {
        if (st.op != S_GEMM || !(st.epi & RDM_EPI_MASK) || st.lmask != RDM_ROW) continue;
        const auto key = std::make_pair(st.mask.id(), norm_lay(g, st.lmask));
        if (!relu_rows.count(key) || g->mbits.count(key)) continue;
        std::vector<uint32_t*> per(ctx->nlocal());
        int64_t ldw = 0;
        for (int sl = 0; sl < ctx->nlocal(); ++sl) {
          const Buf& b = g->bufs[sl].at(key);
          ldw = (b.cols + 31) / 32;
          const size_t bytes = (size_t)std::max<int64_t>(1, b.rows * ldw) * 4;
          g->mem.emplace_back(new DevBuf(bytes));
          per[sl] = g->mem.back()->as<uint32_t>();
          g->ws_bytes += (int64_t)bytes;
        }
        g->mbits[key] = per;
        g->mbits_ld[key] = ldw;
      }
  }
  const int P = ctx->world;
  const int64_t n = g->n_cap;
  g->dwp.assign(ctx->nlocal(), std::vector<float*>(g->L + 1, nullptr));
  g->dbp.assign(ctx->nlocal(), std::vector<float*>(g->L + 1, nullptr));
  g->labels.assign(ctx->nlocal(), nullptr);
  g->mask.assign(ctx->nlocal(), nullptr);
  g->scal.assign(ctx->nlocal(), nullptr);
  for (int s = 0; s < ctx->nlocal(); ++s) {
    const int64_t r = cap_rows(g, ctx->local[s]);
    if (ctx->virtual_group()) {
      for (int l = 1; l <= g->L; ++l) {
        g->mem.emplace_back(new DevBuf((size_t)g->f[l - 1] * g->f[l] * sizeof(float)));
        g->dwp[s][l] = g->mem.back()->as<float>();
        if (g->flags & RDM_GCN_BIAS) {
          g->mem.emplace_back(new DevBuf((size_t)g->f[l] * sizeof(float)));
          g->dbp[s][l] = g->mem.back()->as<float>();
        }
      }
    }
    g->mem.emplace_back(new DevBuf(std::max<int64_t>(r, 1) * sizeof(int32_t)));
    g->labels[s] = g->mem.back()->as<int32_t>();
    g->mem.emplace_back(new DevBuf(std::max<int64_t>(r, 1)));
    g->mask[s] = reinterpret_cast<uint8_t*>(g->mem.back()->ptr);
    g->mem.emplace_back(new DevBuf(4 * sizeof(double)));
    g->scal[s] = reinterpret_cast<double*>(g->mem.back()->ptr);
    RDM_CUDA(cudaMemset(g->scal[s], 0, 4 * sizeof(double)));
  }
  plan_info(pl, g->fwd, g->bwd, n, &g->info, g->RA);
  g->info.workspace_bytes = g->ws_bytes;
  if (ctx->transport == RDM_TRANSPORT_P2P && P > 1 && !g->RA) setup_fusion(g);
  if (!(getenv("RDM_NO_SIDE") && atoi(getenv("RDM_NO_SIDE")))) {
    RDM_CUDA(cudaStreamCreateWithFlags(&g->side, cudaStreamNonBlocking));
    RDM_CUDA(cudaEventCreateWithFlags(&g->ev_fork, cudaEventDisableTiming));
    RDM_CUDA(cudaEventCreateWithFlags(&g->ev_join, cudaEventDisableTiming));
  }
}

// The step after `s` in its pass (nullptr at the end).
const Step* next_step(const rdm_gcn* g, const Step* s) {
  for (auto* v : {&g->fwd, &g->bwd})
    if (!v->empty() && s >= &v->front() && s <= &v->back())
      return s == &v->back() ? nullptr : s + 1;
  return nullptr;
}

void run_step(rdm_gcn* g, const Step& s, const float* const* W) {
  rdm_ctx* ctx = g->ctx;
  // any producer but the bf16-wire redistribution (and the in-place mask,
  // which keeps bf16 values bf16) leaves fp32 values in its output
  if (s.op == S_SPMM || s.op == S_GEMM || s.op == S_LOSS || s.op == S_REDIST) {
    g->wire_bf16.erase({s.out.id(), norm_lay(g, s.lout)});
    g->mb_valid.erase({s.out.id(), norm_lay(g, s.lout)});   // (re)set by the GEMM that writes bits
  }
  const int nl = ctx->nlocal();
  const int P = ctx->world;
  // a fused producer overwrites peers' destination slices: every rank must be
  // done reading their previous contents
  if (s.fuse == 1) p2p_barrier(ctx);
  switch (s.op) {
    case S_SPMM: {
      if (g->RA) {   // Fig. 6: tile broadcast in the column group + row-panel SpMM
        std::vector<const float*> in(nl), mk(nl);
        std::vector<float*> out(nl);
        for (int i = 0; i < nl; ++i) {
          in[i] = buf(g, i, s.in, s.lin).p;
          out[i] = buf(g, i, s.out, s.lout).p;
          mk[i] = (s.epi & RDM_EPI_MASK) ? buf(g, i, s.mask, s.lmask).p : nullptr;
        }
        spmm_panels(ctx, in.data(), out.data(), s.width, s.epi, s.bl ? g->bcur[s.bl - 1] : nullptr,
                    (s.epi & RDM_EPI_MASK) ? mk.data() : nullptr);
        break;
      }
      Phase ph(ctx, RDM_PH_SPMM);
      const Csr& A = s.trans ? g->graph->fwd() : g->graph->bwd();
      for (int i = 0; i < nl; ++i) {
        Buf& in = buf(g, i, s.in, s.lin);
        Buf& out = buf(g, i, s.out, s.lout);
        const float* mk = nullptr;
        int64_t ldm = 0;
        if (s.epi & RDM_EPI_MASK) {
          Buf& m = buf(g, i, s.mask, s.lmask);
          mk = m.p;
          ldm = m.ld;
        }
        const Range cr = P == 1 ? Range{0, s.width} : col_range(s.width, P, ctx->local[i]);
        const int64_t w = cr.size();
        // bias of the column slice (reading R8: added after both products, before σ)
        const float* bias = s.bl ? g->bcur[s.bl - 1] + cr.lo : nullptr;
        ctx->spmm_in_bf16 = g->wire_bf16.count({s.in.id(), norm_lay(g, s.lin)}) > 0;
        if (s.fuse == 1) {
          const Scatter sc = make_scatter(g, s, i);
          spmm(ctx, A, in.p, in.ld, out.p, out.ld, w, s.epi, bias, mk, ldm, &sc);
        } else {
          spmm(ctx, A, in.p, in.ld, out.p, out.ld, w, s.epi, bias, mk, ldm);
        }
        ctx->spmm_in_bf16 = false;
      }
      ctx->counters.spmm_width_units += s.width;
      break;
    }
    case S_GEMM: {
      Phase ph(ctx, RDM_PH_GEMM);
      const int64_t fin = g->f[s.wl - 1], fout = g->f[s.wl];
      // fast variant at P = 1 (row and column layouts coincide): when the next
      // step is an SpMM reading this output, the GEMM's epilogue also writes
      // the SpMM's bf16 input (× s_i for factored values) — the cast folded
      // into the producer (NEXT-3)
      const Step* nxt = next_step(g, &s);
      const bool fold = ctx->prec == RDM_PREC_FAST && P == 1 && nl == 1 && !g->RA && nxt &&
                        nxt->op == S_SPMM && nxt->in.id() == s.out.id() &&
                        !(getenv("RDM_FOLD_CAST") && !atoi(getenv("RDM_FOLD_CAST")));
      for (int i = 0; i < nl; ++i) {
        Buf& in = buf(g, i, s.in, s.lin);
        Buf& out = buf(g, i, s.out, s.lout);
        const float* mk = (s.epi & RDM_EPI_MASK) ? buf(g, i, s.mask, s.lmask).p : nullptr;
        Scatter sc;
        if (s.fuse == 1) sc = make_scatter(g, s, i);
        const int64_t ncol = s.gop == RDM_GEMM_NN ? fout : fin;
        if (fold) {
          const Csr& An = nxt->trans ? g->graph->fwd() : g->graph->bwd();
          const int64_t w8 = (roundup4(ncol) + 7) & ~int64_t(7);
          ctx->gemm_twin = ensure_ws(ctx->ws_bf16, (size_t)std::max<int64_t>(An.in_rows(), 1) * w8 * 2);
          ctx->gemm_twin_ld = w8;
          ctx->gemm_twin_scale = An.fscale ? An.fscale->as<float>() : nullptr;
          ctx->gemm_twin_written = false;
        }
        const auto okey = std::make_pair(s.out.id(), norm_lay(g, s.lout));
        const auto mkey = std::make_pair(s.mask.id(), norm_lay(g, s.lmask));
        auto ob = g->mbits.find(okey);
        if ((s.epi & RDM_EPI_RELU) && ob != g->mbits.end()) {
          ctx->gemm_bits_out = ob->second[i];
          ctx->gemm_bits_ld = g->mbits_ld[okey];
          ctx->gemm_bits_written = false;
        }
        auto mbit = g->mbits.find(mkey);
        if ((s.epi & RDM_EPI_MASK) && mbit != g->mbits.end() && g->mb_valid.count(mkey)) {
          ctx->gemm_mask_bits = mbit->second[i];
          ctx->gemm_mask_bits_ld = g->mbits_ld[mkey];
        }
        gemm(ctx, s.gop, in.p, in.ld, W[s.wl - 1], fout, out.p, out.ld, in.rows, fin, fout, s.epi,
             s.bl ? g->bcur[s.bl - 1] : nullptr, mk, s.fuse == 1 ? &sc : nullptr);
        if (ctx->gemm_bits_out) {
          if (ctx->gemm_bits_written) g->mb_valid.insert(okey);
          else g->mb_valid.erase(okey);
        }
        ctx->gemm_bits_out = nullptr;
        ctx->gemm_mask_bits = nullptr;
        if (fold) {
          ctx->bf16_twin_src = ctx->gemm_twin_written ? out.p : nullptr;
          ctx->bf16_twin_fact = ctx->gemm_twin_scale != nullptr;
          ctx->gemm_twin = nullptr;
          ctx->gemm_twin_scale = nullptr;
        }
      }
      break;
    }
    case S_TN: {
      // fork onto the side stream (inputs are ready on the compute stream);
      // its own split-K workspace, joined in do_backward
      const bool use_side = g->side != nullptr;
      cudaStream_t main = ctx->stream;
      if (use_side) {
        RDM_CUDA(cudaEventRecord(g->ev_fork, main));
        RDM_CUDA(cudaStreamWaitEvent(g->side, g->ev_fork, 0));
        ctx->stream = g->side;
        std::swap(ctx->ws_gemm, g->ws_side);
        g->side_pending = true;
      }
      struct Restore {
        rdm_ctx* c; rdm_gcn* g; cudaStream_t m; bool on;
        ~Restore() { if (on) { c->stream = m; std::swap(c->ws_gemm, g->ws_side); } }
      } restore{ctx, g, main, use_side};
      Phase ph(ctx, RDM_PH_GEMM);
      const int64_t fin = g->f[s.wl - 1], fout = g->f[s.wl];
      for (int i = 0; i < nl; ++i) {
        Buf& x = buf(g, i, s.in, s.lin);
        Buf& u = buf(g, i, s.in2, s.lin2);
        float* dst = g->dwp[i][s.wl];  // per-slot partial, or the caller's dW (set in backward)
        gemm(ctx, RDM_GEMM_TN, x.p, x.ld, u.p, u.ld, dst, fout, x.rows, fin, fout, 0, nullptr,
             nullptr);
      }
      break;
    }
    case S_REDIST: {
      if (s.fuse == 2) {   // the producer already stored it; fence peers before the consumer
        p2p_barrier(ctx);
        count_fused_redist(ctx, (rdm_layout)s.lin, gn(g), s.width);
        break;
      }
      std::vector<const float*> src(nl);
      std::vector<float*> dst(nl);
      for (int i = 0; i < nl; ++i) {
        src[i] = buf(g, i, s.in, s.lin).p;
        dst[i] = buf(g, i, s.out, s.lout).p;
      }
      if (g->RA) {
        redistribute_panels(ctx, (rdm_layout)s.lin, src.data(), dst.data(), gn(g), s.width);
      } else {
        // bf16 wire in the fast variant (NEXT-3) for row → column moves: their
        // destination is an SpMM input, which the fast variant rounds to bf16
        // anyway; column → row moves (SpMM outputs feeding GEMMs and the loss)
        // stay fp32.  RDM_BF16_WIRE=0 disables (experiments).
        const char* wv = getenv("RDM_BF16_WIRE");
        const bool wire = ctx->prec == RDM_PREC_FAST && s.lin == RDM_ROW && P > 1 && !(wv && !atoi(wv));
        redistribute(ctx, (rdm_layout)s.lin, src.data(), dst.data(), gn(g), s.width, wire);
        if (wire) g->wire_bf16.insert({s.out.id(), norm_lay(g, s.lout)});
      }
      break;
    }
    case S_MASK: {
      Phase ph(ctx, RDM_PH_OTHER);
      for (int i = 0; i < nl; ++i) {
        Buf& x = buf(g, i, s.out, s.lout);
        Buf& h = buf(g, i, s.mask, s.lmask);
        apply_mask(ctx, x.p, x.ld, h.p, h.ld, x.rows, x.cols);
      }
      break;
    }
    case S_COLSUM: {   // db^l partial of this slot: 1ᵀ G^l over its rows, at its column offset
      Phase ph(ctx, RDM_PH_OTHER);
      for (int i = 0; i < nl; ++i) {
        Buf& x = buf(g, i, s.in, s.lin);
        float* dst = g->dbp[i][s.bl];
        int64_t lo = 0;
        if (s.lin == RDM_COL && P > 1) {
          if (g->RA) {
            Range r, c;
            int64_t ld;
            tile_of(P, g->RA, gn(g), s.width, ctx->local[i], &r, &c, &ld);
            lo = c.lo;
          } else {
            lo = col_range(s.width, P, ctx->local[i]).lo;
          }
        }
        if (x.cols < s.width) RDM_CUDA(cudaMemsetAsync(dst, 0, s.width * sizeof(float), ctx->stream));
        colsum(ctx, x.p, x.ld, x.rows, x.cols, dst + lo);
      }
      break;
    }
    case S_LOSS: {
      Phase ph(ctx, RDM_PH_LOSS);
      for (int i = 0; i < nl; ++i) {
        Buf& z = buf(g, i, s.in, s.lin);
        Buf& gl = buf(g, i, s.out, s.lout);
        softmax_xent(ctx, z.p, z.ld, g->labels[i], g->mask[i], z.rows, s.width, g->scal[i] + 0,
                     gl.p, gl.ld, g->scal[i] + 1);
      }
      break;
    }
  }
}

std::string step_str(const Step& s) {
  auto k = [](Key x, int l) {
    return std::string(kKindName[x.kind]) + std::to_string(x.layer) + (l == RDM_ROW ? ".row" : ".col");
  };
  std::ostringstream o;
  switch (s.op) {
    case S_SPMM:
      o << "SPMM  " << (s.trans ? "A^T" : "A  ") << " " << k(s.in, s.lin) << " -> " << k(s.out, s.lout)
        << " w=" << s.width << (s.epi & RDM_EPI_RELU ? " +relu" : "")
        << (s.epi & RDM_EPI_MASK ? " *mask(" + k(s.mask, s.lmask) + ")" : "");
      break;
    case S_GEMM:
      o << "GEMM  " << (s.gop == RDM_GEMM_NN ? "NN " : "NT ") << k(s.in, s.lin) << " W" << s.wl << " -> "
        << k(s.out, s.lout) << (s.epi & RDM_EPI_RELU ? " +relu" : "")
        << (s.epi & RDM_EPI_MASK ? " *mask(" + k(s.mask, s.lmask) + ")" : "");
      break;
    case S_TN:
      o << "GEMM  TN " << k(s.in, s.lin) << "^T " << k(s.in2, s.lin2) << " -> Y" << s.wl;
      break;
    case S_REDIST:
      o << "A2A   " << k(s.in, s.lin) << " -> " << k(s.out, s.lout) << " f=" << s.width
        << (s.hidden ? " (hidden)" : "") << (s.fuse == 2 ? " [fused into producer]" : "");
      break;
    case S_MASK:
      o << "MASK  " << k(s.out, s.lout) << " *= 1[" << k(s.mask, s.lmask) << " > 0]";
      break;
    case S_LOSS:
      o << "LOSS  " << k(s.in, s.lin) << " -> " << k(s.out, s.lout);
      break;
    case S_COLSUM:
      o << "BSUM  1^T " << k(s.in, s.lin) << " -> db" << s.bl;
      break;
  }
  if ((s.op == S_SPMM || s.op == S_GEMM) && s.bl) o << " +b" << s.bl;
  return o.str();
}

std::string describe_steps(const std::vector<Step>& fwd, const std::vector<Step>& bwd) {
  std::string s = "forward:\n";
  for (auto& st : fwd) s += "  " + step_str(st) + "\n";
  s += "backward:\n";
  for (auto& st : bwd) s += "  " + step_str(st) + "\n";
  return s;
}

struct FwdArgs {
  rdm_gcn* g;
  const float* const* W;
  const float* const* b;
  double* loss;
};
struct BwdArgs {
  rdm_gcn* g;
  const float* const* W;
  float* const* dW;
  float* const* db;
};

void consume_staged(rdm_gcn* g);

void do_forward(void* a_) {
  auto* a = static_cast<FwdArgs*>(a_);
  rdm_gcn* g = a->g;
  rdm_ctx* ctx = g->ctx;
  sync_graph(g);
  if (!g->input_set) throw Error(RDM_ERR_STATE, "rdm_gcn_forward: call rdm_gcn_set_input first");
  RDM_CHECK_ARG(a->W && a->loss, "rdm_gcn_forward: W and loss_dev required");
  for (int l = 0; l < g->L; ++l) RDM_CHECK_ARG(a->W[l], "rdm_gcn_forward: null W");
  const bool bias = (g->flags & RDM_GCN_BIAS) != 0;
  RDM_CHECK_ARG(!bias || a->b, "rdm_gcn_forward: the model has biases (RDM_GCN_BIAS): b required");
  if (bias)
    for (int l = 0; l < g->L; ++l) RDM_CHECK_ARG(a->b[l], "rdm_gcn_forward: null b");
  g->bcur = bias ? a->b : nullptr;
  if (g->staged) {
    Phase ph(ctx, RDM_PH_OTHER);
    consume_staged(g);
  }
  for (auto& s : g->fwd) run_step(g, s, a->W);
  g->bcur = nullptr;
  const int nl = ctx->nlocal();
  std::vector<double*> parts(nl);
  for (int i = 0; i < nl; ++i) parts[i] = g->scal[i] + 1;
  allreduce_d(ctx, parts.data(), 1);
  {
    Phase ph(ctx, RDM_PH_LOSS);
    finish_loss(ctx, g->scal[0] + 1, g->scal[0] + 0, a->loss);
  }
  if (g->saint && g->saint->ev_free[g->sbuf]) {   // forward-only use also releases the buffer
    RDM_CUDA(cudaEventRecord(g->saint->ev_free[g->sbuf], ctx->stream));
    g->saint->freed[g->sbuf] = true;
  }
}

void do_backward(void* a_) {
  auto* a = static_cast<BwdArgs*>(a_);
  rdm_gcn* g = a->g;
  rdm_ctx* ctx = g->ctx;
  RDM_CHECK_ARG(a->W && a->dW, "rdm_gcn_backward: W and dW required");
  if (g->saint && g->gver != g->saint->version)
    throw Error(RDM_ERR_STATE, "rdm_gcn_backward: the subgraph changed since the forward pass");
  for (int l = 0; l < g->L; ++l) RDM_CHECK_ARG(a->W[l] && a->dW[l], "rdm_gcn_backward: null W/dW");
  const bool bias = (g->flags & RDM_GCN_BIAS) != 0;
  RDM_CHECK_ARG(!bias || a->db, "rdm_gcn_backward: the model has biases (RDM_GCN_BIAS): db required");
  if (bias)
    for (int l = 0; l < g->L; ++l) RDM_CHECK_ARG(a->db[l], "rdm_gcn_backward: null db");
  if (!ctx->virtual_group())
    for (int l = 1; l <= g->L; ++l) {
      g->dwp[0][l] = a->dW[l - 1];
      if (bias) g->dbp[0][l] = a->db[l - 1];
    }
  for (auto& s : g->bwd) run_step(g, s, a->W);
  if (g->side_pending) {   // every weight gradient is in place before the reduction
    RDM_CUDA(cudaEventRecord(g->ev_join, g->side));
    RDM_CUDA(cudaStreamWaitEvent(ctx->stream, g->ev_join, 0));
    g->side_pending = false;
  }
  if (g->saint && g->saint->ev_free[g->sbuf]) {   // the sampler may rebuild this buffer now
    RDM_CUDA(cudaEventRecord(g->saint->ev_free[g->sbuf], ctx->stream));
    g->saint->freed[g->sbuf] = true;
  }
  const int nl = ctx->nlocal();
  for (int l = 1; l <= g->L; ++l) {
    const int64_t cnt = g->f[l - 1] * g->f[l];
    if (ctx->virtual_group()) {
      Phase ph(ctx, RDM_PH_ALLREDUCE);
      std::vector<const float*> parts(nl);
      for (int i = 0; i < nl; ++i) parts[i] = g->dwp[i][l];
      sum_slots(ctx, a->dW[l - 1], parts.data(), nl, cnt);
      ctx->counters.allreduce_bytes += cnt * 4;
    } else {
      float* b = a->dW[l - 1];
      allreduce(ctx, &b, cnt);
    }
    if (bias) {   // db^l: the slots' partials (row slices / column ranges) summed like Y^l
      if (ctx->virtual_group()) {
        Phase ph(ctx, RDM_PH_ALLREDUCE);
        std::vector<const float*> parts(nl);
        for (int i = 0; i < nl; ++i) parts[i] = g->dbp[i][l];
        sum_slots(ctx, a->db[l - 1], parts.data(), nl, g->f[l]);
        ctx->counters.allreduce_bytes += g->f[l] * 4;
      } else {
        float* b = a->db[l - 1];
        allreduce(ctx, &b, g->f[l]);
      }
    }
  }
}

struct InputArgs {
  rdm_gcn* g;
  const float* const* H0;
  const int32_t* const* labels;
  const uint8_t* const* mask;
  int on_host;
};

// Host inputs are double-buffered: rdm_gcn_set_input(on_host) only enqueues
// the H2D copy into device staging buffers on a private copy stream (after the
// previous input has been consumed) and returns; the next rdm_gcn_forward
// makes the compute stream wait for it and moves the staged input into place
// (D2D).  The next step's 0.5 GB input copy therefore overlaps the current
// step's compute instead of serialising with it.
void stage_host_input(rdm_gcn* g, const InputArgs* a) {
  rdm_ctx* ctx = g->ctx;
  const int nl = ctx->nlocal(), P = ctx->world;
  const int64_t n = gn(g), f0 = g->f[0];
  RDM_CHECK_ARG(!g->saint, "set_input: a sampler's GCN takes rdm_saint_set_input");
  if (!g->cs) {
    RDM_CUDA(cudaStreamCreateWithFlags(&g->cs, cudaStreamNonBlocking));
    RDM_CUDA(cudaEventCreateWithFlags(&g->ev_ready, cudaEventDisableTiming));
    RDM_CUDA(cudaEventCreateWithFlags(&g->ev_free, cudaEventDisableTiming));
    g->st_h0.assign(nl, nullptr);
    g->st_lab.assign(nl, nullptr);
    g->st_mask.assign(nl, nullptr);
    for (int i = 0; i < nl; ++i) {
      const int64_t r = row_range(n, P, ctx->local[i]).size();
      g->mem.emplace_back(new DevBuf((size_t)std::max<int64_t>(1, r * f0) * sizeof(float)));
      g->st_h0[i] = g->mem.back()->as<float>();
      g->mem.emplace_back(new DevBuf((size_t)std::max<int64_t>(1, r) * sizeof(int32_t)));
      g->st_lab[i] = g->mem.back()->as<int32_t>();
      g->mem.emplace_back(new DevBuf((size_t)std::max<int64_t>(1, r)));
      g->st_mask[i] = reinterpret_cast<uint8_t*>(g->mem.back()->ptr);
    }
  }
  RDM_CUDA(cudaStreamWaitEvent(g->cs, g->ev_free, 0));   // previous staged input consumed
  for (int i = 0; i < nl; ++i) {
    const int64_t r = row_range(n, P, ctx->local[i]).size();
    if (!r) continue;
    if (f0)
      RDM_CUDA(cudaMemcpyAsync(g->st_h0[i], a->H0[i], r * f0 * sizeof(float), cudaMemcpyHostToDevice, g->cs));
    RDM_CUDA(cudaMemcpyAsync(g->st_lab[i], a->labels[i], r * sizeof(int32_t), cudaMemcpyHostToDevice, g->cs));
    if (a->mask && a->mask[i])
      RDM_CUDA(cudaMemcpyAsync(g->st_mask[i], a->mask[i], r, cudaMemcpyHostToDevice, g->cs));
    else
      RDM_CUDA(cudaMemsetAsync(g->st_mask[i], 1, r, g->cs));
  }
  RDM_CUDA(cudaEventRecord(g->ev_ready, g->cs));
  g->staged = true;
  g->input_set = true;
}

void apply_input(rdm_gcn* g, const InputArgs* a);

// Called at the start of forward: consume a staged host input on the compute stream.
void consume_staged(rdm_gcn* g) {
  if (!g->staged) return;
  rdm_ctx* ctx = g->ctx;
  RDM_CUDA(cudaStreamWaitEvent(ctx->stream, g->ev_ready, 0));
  const int nl = ctx->nlocal();
  std::vector<const float*> h(g->st_h0.begin(), g->st_h0.end());
  std::vector<const int32_t*> l(g->st_lab.begin(), g->st_lab.end());
  std::vector<const uint8_t*> m(g->st_mask.begin(), g->st_mask.end());
  (void)nl;
  InputArgs a{g, h.data(), l.data(), m.data(), 0};
  apply_input(g, &a);           // device-to-device into the working buffers
  RDM_CUDA(cudaEventRecord(g->ev_free, ctx->stream));
  g->staged = false;
}

void do_set_input(void* a_) {
  auto* a = static_cast<InputArgs*>(a_);
  rdm_gcn* g = a->g;
  RDM_CHECK_ARG(a->H0 && a->labels, "set_input: H0 and labels required");
  if (a->on_host) {
    stage_host_input(g, a);
  } else {
    g->staged = false;
    apply_input(g, a);
  }
}

void apply_input(rdm_gcn* g, const InputArgs* a) {
  rdm_ctx* ctx = g->ctx;
  const int nl = ctx->nlocal(), P = ctx->world;
  const int64_t n = gn(g), f0 = g->f[0];
  RDM_CHECK_ARG(!g->saint, "set_input: a sampler's GCN takes rdm_saint_set_input");
  const cudaMemcpyKind kind = a->on_host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  const rdm_counters saved = ctx->counters;
  std::vector<const float*> src(nl);
  std::vector<float*> dst(nl);
  for (int i = 0; i < nl; ++i) {
    const int64_t r = row_range(n, P, ctx->local[i]).size();
    Buf& h = buf(g, i, {K_H, 0}, RDM_ROW);
    if (r && f0) {
      if (h.ld == f0) {
        RDM_CUDA(cudaMemcpyAsync(h.p, a->H0[i], r * f0 * sizeof(float), kind, ctx->stream));
      } else if (!a->on_host) {
        copy_2d(ctx, h.p, h.ld, a->H0[i], f0, r, f0);   // device source: re-pitch directly
      } else {
        // one contiguous (DMA-friendly) copy, then re-pitch to ld on the device
        float* stage = ensure_ws(ctx->ws_stage, (size_t)r * f0 * sizeof(float));
        RDM_CUDA(cudaMemcpyAsync(stage, a->H0[i], r * f0 * sizeof(float), kind, ctx->stream));
        copy_2d(ctx, h.p, h.ld, stage, f0, r, f0);
      }
    }
    if (r) {
      RDM_CUDA(cudaMemcpyAsync(g->labels[i], a->labels[i], r * sizeof(int32_t), kind, ctx->stream));
      if (a->mask && a->mask[i])
        RDM_CUDA(cudaMemcpyAsync(g->mask[i], a->mask[i], r, kind, ctx->stream));
      else
        RDM_CUDA(cudaMemsetAsync(g->mask[i], 1, r, ctx->stream));
    }
    src[i] = h.p;
    auto hc = g->bufs[i].find({Key{K_H, 0}.id(), norm_lay(g, RDM_COL)});
    dst[i] = hc == g->bufs[i].end() ? nullptr : hc->second.p;
  }
  // H^0's column slices only if the plan reads them (reading R12)
  const bool need_col = P > 1 && dst[0] != nullptr;
  if (need_col && g->RA)
    redistribute_panels(ctx, RDM_ROW, src.data(), dst.data(), n, f0);
  else if (need_col)
    redistribute(ctx, RDM_ROW, src.data(), dst.data(), n, f0);
  std::vector<double*> nt(nl);
  for (int i = 0; i < nl; ++i) {
    const int64_t r = row_range(n, P, ctx->local[i]).size();
    count_mask(ctx, g->mask[i], r, g->scal[i] + 0);
    nt[i] = g->scal[i] + 0;
  }
  allreduce_d(ctx, nt.data(), 1);
  ctx->counters = saved;
  g->input_set = true;
}


struct SaintInputArgs {
  rdm_gcn* g;
  const float* H;
  int64_t ldh;
  const int32_t* labels;
  const uint8_t* mask;
};

// GraphSAINT input: gathered on the device from the full-graph arrays every
// rank holds — H^0 straight into both layouts, so no redistribution.
void do_saint_input(void* a_) {
  auto* a = static_cast<SaintInputArgs*>(a_);
  rdm_gcn* g = a->g;
  rdm_ctx* ctx = g->ctx;
  RDM_CHECK_ARG(g->saint, "rdm_saint_set_input: not a sampler's GCN (rdm_saint_gcn_create)");
  RDM_CHECK_ARG(a->H && a->labels && a->ldh >= g->f[0], "rdm_saint_set_input: bad arguments");
  sync_graph(g);
  Phase ph(ctx, RDM_PH_SAMPLE);
  const int P = ctx->world;
  const int64_t n = gn(g), f0 = g->f[0];
  const int32_t* nodes = g->saint->nodes_b[g->sbuf]->as<int32_t>();
  for (int i = 0; i < ctx->nlocal(); ++i) {
    const int p = ctx->local[i];
    const Range r = row_range(n, P, p);
    Buf& hr = buf(g, i, {K_H, 0}, RDM_ROW);
    saint_gather(ctx, a->H, a->ldh, nodes, r.lo, r.size(), 0, f0, hr.p, hr.ld);
    auto hc = g->bufs[i].find({Key{K_H, 0}.id(), norm_lay(g, RDM_COL)});
    if (P > 1 && hc != g->bufs[i].end()) {
      const Range c = col_range(f0, P, p);
      saint_gather(ctx, a->H, a->ldh, nodes, 0, n, c.lo, c.size(), hc->second.p, hc->second.ld);
    }
    saint_gather_labels(ctx, a->labels, a->mask, nodes, r.lo, r.size(), g->labels[i], g->mask[i]);
  }
  // the subgraph's training count from the whole node list (no communication)
  uint8_t* ms = reinterpret_cast<uint8_t*>(ensure_ws(g->saint->mask_s, std::max<int64_t>(n, 1)));
  saint_gather_labels(ctx, a->labels, a->mask, nodes, 0, n, nullptr, ms);
  for (int i = 0; i < ctx->nlocal(); ++i) count_mask(ctx, ms, n, g->scal[i] + 0);
  g->staged = false;
  g->input_set = true;
}

void do_create(void* a_) { create(static_cast<rdm_gcn*>(a_)); }

}  // namespace
}  // namespace rdm

extern "C" {

rdm_status rdm_gcn_create(rdm_ctx* ctx, int L, const int64_t* f, const rdm_config* cfg, int flags,
                          rdm_gcn** out) {
  if (!ctx || !out || !f || !cfg || L < 1 || L > RDM_MAX_LAYERS || cfg->L != L) return RDM_ERR_ARG;
  for (int l = 0; l <= L; ++l)
    if (f[l] < 1) return RDM_ERR_ARG;
  const bool panels = (flags & RDM_GCN_PANELS) != 0;
  if (panels && ctx->panel_RA <= 0) {
    ctx->err = "rdm_gcn_create: RDM_GCN_PANELS needs rdm_set_graph_panels";
    return RDM_ERR_STATE;
  }
  if (!panels && !ctx->has_graph) {
    ctx->err = "rdm_gcn_create: no graph (call rdm_set_graph)";
    return RDM_ERR_STATE;
  }
  auto* g = new rdm_gcn();
  g->ctx = ctx;
  g->graph = panels ? nullptr : &ctx->graph;
  g->n_cap = panels ? ctx->panel_n : ctx->graph.n;
  g->RA = panels ? ctx->panel_RA : 0;
  g->L = L;
  g->flags = flags;
  g->f.assign(f, f + L + 1);
  g->cfg = *cfg;
  rdm_status st = rdm_guarded_call(ctx, do_create, g);
  if (st != RDM_OK) {
    delete g;
    return st;
  }
  *out = g;
  return RDM_OK;
}

rdm_status rdm_saint_gcn_create(rdm_saint* s, int L, const int64_t* f, const rdm_config* cfg,
                                int flags, rdm_gcn** out) {
  if (!s || !out || !f || !cfg || L < 1 || L > RDM_MAX_LAYERS || cfg->L != L) return RDM_ERR_ARG;
  rdm_ctx* ctx = s->ctx;
  for (int l = 0; l <= L; ++l)
    if (f[l] < 1) return RDM_ERR_ARG;
  auto* g = new rdm_gcn();
  g->ctx = ctx;
  g->graph = &s->graph();
  g->saint = s;
  g->n_cap = s->n_cap;
  g->L = L;
  g->flags = flags;
  g->f.assign(f, f + L + 1);
  g->cfg = *cfg;
  rdm_status st = rdm_guarded_call(ctx, do_create, g);
  if (st != RDM_OK) {
    delete g;
    return st;
  }
  *out = g;
  return RDM_OK;
}

rdm_status rdm_saint_set_input(rdm_gcn* g, const float* H0_full, int64_t ld_h,
                               const int32_t* labels_full, const uint8_t* mask_full) {
  if (!g) return RDM_ERR_ARG;
  SaintInputArgs a{g, H0_full, ld_h, labels_full, mask_full};
  return rdm_guarded_call(g->ctx, do_saint_input, &a);
}

rdm_status rdm_gcn_destroy(rdm_gcn* g) {
  if (!g) return RDM_ERR_ARG;
  cudaSetDevice(g->ctx->device);
  cudaStreamSynchronize(g->ctx->stream);
  if (g->cs) {
    cudaStreamSynchronize(g->cs);
    cudaStreamDestroy(g->cs);
    cudaEventDestroy(g->ev_ready);
    cudaEventDestroy(g->ev_free);
  }
  if (g->side) {
    cudaStreamSynchronize(g->side);
    cudaStreamDestroy(g->side);
    cudaEventDestroy(g->ev_fork);
    cudaEventDestroy(g->ev_join);
  }
  if (!g->ipc_opened.empty()) {
    // no rank may free a slice a peer still maps: close, then fence, then free
    for (void* p : g->ipc_opened) cudaIpcCloseMemHandle(p);
    rdm_guarded_call(g->ctx, [](void* c) { p2p_barrier(static_cast<rdm_ctx*>(c)); }, g->ctx);
    cudaStreamSynchronize(g->ctx->stream);
  }
  delete g;
  return RDM_OK;
}

rdm_status rdm_gcn_set_input(rdm_gcn* g, const float* const* H0_row, const int32_t* const* labels_row,
                             const uint8_t* const* mask_row, int on_host) {
  if (!g) return RDM_ERR_ARG;
  InputArgs a{g, H0_row, labels_row, mask_row, on_host};
  return rdm_guarded_call(g->ctx, do_set_input, &a);
}

rdm_status rdm_gcn_forward(rdm_gcn* g, const float* const* W, const float* const* b,
                           double* loss_dev) {
  if (!g) return RDM_ERR_ARG;
  FwdArgs a{g, W, b, loss_dev};
  return rdm_guarded_call(g->ctx, do_forward, &a);
}

rdm_status rdm_gcn_backward(rdm_gcn* g, const float* const* W, float* const* dW, float* const* db) {
  if (!g) return RDM_ERR_ARG;
  BwdArgs a{g, W, dW, db};
  return rdm_guarded_call(g->ctx, do_backward, &a);
}

rdm_status rdm_gcn_tensor(rdm_gcn* g, int which, int layer, int slot, rdm_layout layout,
                          const float** ptr, int64_t* rows, int64_t* cols, int64_t* ld) {
  if (!g || slot < 0 || slot >= g->ctx->nlocal()) return RDM_ERR_ARG;
  Key k;
  switch (which) {
    case RDM_T_H: k = {K_H, layer}; break;
    case RDM_T_Z: k = {K_Z, 0}; break;
    case RDM_T_G: k = {K_G, layer}; break;
    case RDM_T_MEMO: k = {K_T, layer}; break;
    case RDM_T_DWP: {
      if (layer < 1 || layer > g->L || !g->dwp[slot][layer]) return RDM_ERR_ARG;
      if (ptr) *ptr = g->dwp[slot][layer];
      if (rows) *rows = g->f[layer - 1];
      if (cols) *cols = g->f[layer];
      if (ld) *ld = g->f[layer];
      return RDM_OK;
    }
    default: return RDM_ERR_ARG;
  }
  if (which == RDM_T_MEMO && (layer < 1 || layer > g->L || g->cfg.fwd_D[layer - 1])) return RDM_ERR_ARG;
  auto it = g->bufs[slot].find({k.id(), norm_lay(g, layout)});
  if (it == g->bufs[slot].end()) {
    g->ctx->err = "rdm_gcn_tensor: tensor not resident in that layout";
    return RDM_ERR_ARG;
  }
  const Buf& b = it->second;
  if (!b.valid_end) {
    g->ctx->err = "rdm_gcn_tensor: RDM_GCN_LOW_MEMORY reuses this tensor's memory later in the epoch";
    return RDM_ERR_STATE;
  }
  if (ptr) *ptr = b.p;
  if (rows) *rows = b.rows;
  if (cols) *cols = b.cols;
  if (ld) *ld = b.ld;
  return RDM_OK;
}

rdm_status rdm_gcn_get_info(const rdm_gcn* g, rdm_gcn_info* out) {
  if (!g || !out) return RDM_ERR_ARG;
  *out = g->info;
  return RDM_OK;
}

rdm_status rdm_gcn_describe(const rdm_gcn* g, char* buf, size_t cap) {
  if (!g || !buf || !cap) return RDM_ERR_ARG;
  const std::string s = describe_steps(g->fwd, g->bwd);
  std::snprintf(buf, cap, "%s", s.c_str());
  return s.size() < cap ? RDM_OK : RDM_ERR_ARG;
}

}  // extern "C"

extern "C" rdm_status rdm_plan_info(int L, const int64_t* f, const rdm_config* cfg, int P, int64_t n,
                                    int flags, rdm_gcn_info* out, char* desc, size_t cap) {
  if (L < 1 || L > RDM_MAX_LAYERS || !f || !cfg || cfg->L != L || P < 1 || n < 0) return RDM_ERR_ARG;
  try {
    Planner pl;
    pl.L = L;
    pl.P = P;
    pl.f.assign(f, f + L + 1);
    pl.cfg = *cfg;
    pl.igrad = (flags & RDM_GCN_INPUT_GRAD) != 0;
    pl.bias = (flags & RDM_GCN_BIAS) != 0;
    std::vector<Step> fwd, bwd;
    pl.plan(fwd, bwd);
    if (out) {
      plan_info(pl, fwd, bwd, n, out);
      // activation workspace of rank 0 (full replication, no sampler)
      ShapeCtx sc;
      sc.P = P;
      sc.n_cap = n;
      std::vector<BufPlan> bp = buffer_lifetimes(pl, fwd, bwd);
      int64_t bytes = 0;
      for (const SlabPlan& sl : plan_slabs(bp, sc, (flags & RDM_GCN_LOW_MEMORY) != 0)) bytes += (int64_t)sl.bytes;
      out->workspace_bytes = bytes;
    }
    if (desc && cap) {
      const std::string s = describe_steps(fwd, bwd);
      std::snprintf(desc, cap, "%s", s.c_str());
      if (s.size() >= cap) return RDM_ERR_ARG;
    }
    return RDM_OK;
  } catch (const std::exception&) {
    return RDM_ERR_STATE;
  }
}
