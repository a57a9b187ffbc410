// plan.cpp — the paper's configuration cost model and selector (host).
//
// PAPER.md §IV (L175-224), Tables II-IV, Table VI:
//   * a redistribution of an N x f matrix moves (P−1)/P·N·f elements (L142);
//     the model counts its width f (unit (P−1)/P·N, L224);
//   * an SpMM on an N x f operand is nnz·f FMAs (L142); the model counts f;
//   * SpMM needs column slices, GEMM row slices (§III-A), so each layer
//     pays one redistribution of its intermediate (L140) plus whatever its
//     neighbours leave in the wrong layout (L210); the loss needs row slices
//     (L206); backward mirrors forward (L208, Table III) and a GEMM-first
//     backward layer without the forward memo AᵀH^{l-1} (L118-127) pays an
//     extra SpMM of width min(f_{l-1}, f_l) and 2·min of redistribution
//     (Table III N.M. rows);
//   * H^0 is available in both layouts (IDs 2/3/10 of Table IV carry no f_in).
// Pareto filter on (comm, sparse) (L31, L224) and a pick among the front.
#include <algorithm>
#include <cmath>

#include "internal.h"

namespace rdm {

int64_t config_to_id(const rdm_config& c) {
  int64_t v = 0;
  for (int l = c.L; l >= 1; --l) v = (v << 1) | (c.bwd_D[l - 1] ? 1 : 0);
  for (int l = 1; l <= c.L; ++l) v = (v << 1) | (c.fwd_D[l - 1] ? 1 : 0);
  return v;
}

rdm_config config_from_id(int L, int64_t id) {
  rdm_config c{};
  c.L = L;
  // LSB side holds fwd L ... fwd 1 (fwd L is bit 0), then bwd 1 ... bwd L
  for (int l = L; l >= 1; --l) {
    c.fwd_D[l - 1] = (uint8_t)(id & 1);
    id >>= 1;
  }
  for (int l = 1; l <= L; ++l) {
    c.bwd_D[l - 1] = (uint8_t)(id & 1);
    id >>= 1;
  }
  return c;
}

// Layout-tracking evaluation of Tables II/III rules.  bit 1 = row, bit 2 = col.
void model_costs(int L, const int64_t* f, int need_input_grad, const rdm_config& c, int64_t* comm_out,
                 int64_t* sparse_out) {
  enum { R = 1, C = 2 };
  int64_t comm = 0, sparse = 0;
  std::vector<int> H(L + 1, 0), G(L + 1, 0);
  std::vector<bool> memo(L + 1, false);
  H[0] = R | C;
  for (int l = 1; l <= L; ++l) {
    if (!c.fwd_D[l - 1]) {  // SpMM first: T = Aᵀ H^{l-1} (col) → row, Z = T W
      if (!(H[l - 1] & C)) { comm += f[l - 1]; H[l - 1] |= C; }
      sparse += f[l - 1];
      comm += f[l - 1];
      memo[l] = true;
      H[l] = R;
    } else {                // GEMM first: T = H W (row) → col, Z = Aᵀ T
      if (!(H[l - 1] & R)) { comm += f[l - 1]; H[l - 1] |= R; }
      comm += f[l];
      sparse += f[l];
      H[l] = C;
    }
  }
  if (!(H[L] & R)) comm += f[L];  // loss needs rows whole (L206)
  G[L] = R;
  for (int l = L; l >= 1; --l) {
    const bool out = (l > 1) || need_input_grad;
    if (!c.bwd_D[l - 1]) {  // U = A G^l (col) → row; Y = H^{l-1}ᵀ U; G^{l-1} = U Wᵀ
      if (!(G[l] & C)) { comm += f[l]; G[l] |= C; }
      sparse += f[l];
      comm += f[l];
      G[l - 1] = R;
    } else {                // V = G^l Wᵀ (row) → col; G^{l-1} = A V; Y = T_lᵀ G^l
      if (!(G[l] & R)) { comm += f[l]; G[l] |= R; }
      if (out) {
        comm += f[l - 1];
        sparse += f[l - 1];
      }
      G[l - 1] = C;
      if (!memo[l]) {
        const int64_t mn = std::min(f[l - 1], f[l]);
        sparse += mn;
        comm += 2 * mn;
      }
    }
  }
  *comm_out = comm;
  *sparse_out = sparse;
}

}  // namespace rdm

using namespace rdm;

extern "C" {

rdm_status rdm_config_from_id(int L, int64_t id, rdm_config* out) {
  if (L < 1 || L > RDM_MAX_LAYERS || !out || id < 0 || id >= (int64_t(1) << (2 * L)))
    return RDM_ERR_ARG;
  *out = config_from_id(L, id);
  return RDM_OK;
}

int64_t rdm_config_to_id(const rdm_config* cfg) { return cfg ? config_to_id(*cfg) : -1; }

rdm_status rdm_config_costs(int L, const int64_t* f, int need_input_grad, int64_t id,
                            int64_t* comm_units, int64_t* sparse_units) {
  if (L < 1 || L > RDM_MAX_LAYERS || !f || id < 0 || id >= (int64_t(1) << (2 * L)))
    return RDM_ERR_ARG;
  int64_t c, s;
  model_costs(L, f, need_input_grad, config_from_id(L, id), &c, &s);
  if (comm_units) *comm_units = c;
  if (sparse_units) *sparse_units = s;
  return RDM_OK;
}

rdm_status rdm_select_config(int L, const int64_t* f, int64_t n, int64_t nnz, int P,
                             int need_input_grad, int64_t* pareto_ids, int* n_pareto,
                             int64_t* chosen_id, int64_t* comm_units, int64_t* sparse_units) {
  if (L < 1 || L > 6 || !f || P < 1 || n < 0 || nnz < 0) return RDM_ERR_ARG;
  const int64_t ncfg = int64_t(1) << (2 * L);
  std::vector<int64_t> cc(ncfg), ss(ncfg);
  for (int64_t i = 0; i < ncfg; ++i) model_costs(L, f, need_input_grad, config_from_id(L, i), &cc[i], &ss[i]);
  std::vector<int64_t> front;
  for (int64_t i = 0; i < ncfg; ++i) {
    bool dom = false;
    for (int64_t j = 0; j < ncfg && !dom; ++j)
      dom = cc[j] <= cc[i] && ss[j] <= ss[i] && (cc[j] < cc[i] || ss[j] < ss[i]);
    if (!dom) front.push_back(i);
  }
  if (n_pareto) {
    const int cap = *n_pareto;
    for (int k = 0; k < (int)front.size() && k < cap && pareto_ids; ++k) pareto_ids[k] = front[k];
    *n_pareto = (int)front.size();
  }
  // Pick (reading R23): modelled B200 time.  Redistribution: each unit of
  // width moves (P−1)/P·N·4 bytes total, i.e. (P−1)/P²·N·4 per GPU, over
  // NVLink at 770 GB/s per direction (the peer-copy bandwidth
  // B200_PROFILING.md reports for this pool; not measured by this build —
  // every box it ran on had one GPU).  SpMM: each call streams the
  // replicated CSR (≈8 B/nnz + 8 B/row) and its N x w/P slice twice
  // (≈6.5 TB/s HBM).  The number of SpMM calls is not in the model; the
  // width term is what the paper's sparse units measure.
  const double B_link = 770e9, B_hbm = 6.5e12;
  int64_t best = -1;
  double best_t = 0;
  for (int64_t i : front) {
    const double comm_bytes = P > 1 ? (double)cc[i] * (P - 1) / ((double)P * P) * n * 4.0 : 0.0;
    const double spmm_bytes = (double)ss[i] * ((double)nnz * 4.0 / P + 8.0 * n / P);
    const double t = comm_bytes / B_link + spmm_bytes / B_hbm;
    if (best < 0 || t < best_t * (1 - 1e-12) ||
        (std::fabs(t - best_t) <= 1e-12 * best_t && (ss[i] < ss[best] || (ss[i] == ss[best] && i < best)))) {
      best = i;
      best_t = t;
    }
  }
  if (chosen_id) *chosen_id = best;
  if (comm_units) *comm_units = best >= 0 ? cc[best] : 0;
  if (sparse_units) *sparse_units = best >= 0 ? ss[best] : 0;
  return RDM_OK;
}

}  // extern "C"

// R_A < P (§III-E; reading R35): elements moved per epoch by a configuration
// = N·[(R_A−1)/R_A·comm_units + (P/R_A−1)·sparse_units]; Pareto in (elements,
// sparse units); the pick adds the same B200 time model as rdm_select_config
// with the elements spread over P GPUs.
extern "C" rdm_status rdm_select_config_ra(int L, const int64_t* f, int64_t n, int64_t nnz, int P,
                                           int R_A, int need_input_grad, int64_t* pareto_ids,
                                           int* n_pareto, int64_t* chosen_id, double* comm_elems,
                                           int64_t* sparse_units) {
  if (L < 1 || L > 6 || !f || P < 1 || R_A < 1 || R_A > P || P % R_A || n < 0 || nnz < 0)
    return RDM_ERR_ARG;
  const int64_t ncfg = int64_t(1) << (2 * L);
  std::vector<double> ce(ncfg);
  std::vector<int64_t> ss(ncfg);
  for (int64_t i = 0; i < ncfg; ++i) {
    int64_t c, sp;
    model_costs(L, f, need_input_grad, config_from_id(L, i), &c, &sp);
    ce[i] = (double)n * ((double)(R_A - 1) / R_A * c + ((double)P / R_A - 1) * sp);
    ss[i] = sp;
  }
  std::vector<int64_t> front;
  for (int64_t i = 0; i < ncfg; ++i) {
    bool dom = false;
    for (int64_t j = 0; j < ncfg && !dom; ++j)
      dom = ce[j] <= ce[i] && ss[j] <= ss[i] && (ce[j] < ce[i] || ss[j] < ss[i]);
    if (!dom) front.push_back(i);
  }
  if (n_pareto) {
    const int cap = *n_pareto;
    for (int k = 0; k < (int)front.size() && k < cap && pareto_ids; ++k) pareto_ids[k] = front[k];
    *n_pareto = (int)front.size();
  }
  const double B_link = 770e9, B_hbm = 6.5e12;
  int64_t best = -1;
  double best_t = 0;
  for (int64_t i : front) {
    const double t = ce[i] * 4.0 / P / B_link + (double)ss[i] * ((double)nnz * 4.0 / P + 8.0 * n / P) / B_hbm;
    if (best < 0 || t < best_t * (1 - 1e-12) ||
        (std::fabs(t - best_t) <= 1e-12 * best_t && (ss[i] < ss[best] || (ss[i] == ss[best] && i < best)))) {
      best = i;
      best_t = t;
    }
  }
  if (chosen_id) *chosen_id = best;
  if (comm_elems) *comm_elems = best >= 0 ? ce[best] : 0.0;
  if (sparse_units) *sparse_units = best >= 0 ? ss[best] : 0;
  return RDM_OK;
}
