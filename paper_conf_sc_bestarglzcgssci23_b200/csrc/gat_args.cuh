// gat_args.cuh — argument blocks shared by the GAT sparse kernels (gat.cu, gat_k128.cu)
#pragma once
#include "internal.cuh"

namespace agnn {

struct GatFwdOut {
  float* Z;      // [n_local x K]   nullable (inference)
  float* Hout;   // [n_local x K]
  float* m;      // [n_local x NH]  nullable
  float* l;      // [n_local x NH]  nullable
  float* pacc;   // [n_chunks x K]
  float* pm;     // [n_chunks x NH]
  float* pl;     // [n_chunks x NH]
  // factored backward (gat_factored()): Q_i = sum_j c_ij P_j - (sum_j c_ij) Z_i with
  // c_ij = alpha_ij lambda_ij, so that ds_i = G_i . Q_i (per head) needs no gathers
  float* Q;      // [n_local x K]   nullable (inference, or the unfactored path)
  float* pu;     // [n_chunks x K]  chunk partials of sum_j p_ij lambda_ij P_j
  float* pc;     // [n_chunks x NH] chunk partials of sum_j p_ij lambda_ij
};

struct GatBwdArgs {
  const float* P;      // [n_tot x K]
  const float* st;     // [n_tot x 2NH]   (s | t)
  const float* G;      // [n_tot x K]
  const float4* rec;   // [n_tot x NH]    {s, m, 1/l, delta}
  const float* a;      // [NH x 2D]
  float slope;
  float* dP;           // [n_local x K]
  float* pacc;         // [n_chunks x 3K] heavy-row chunk partials
  float* pds;          // [n_chunks x NH]
  float* pdt;          // [n_chunks x NH]
  float* da_part;      // [warps x 2K]
  float* ds_out;       // [n_local x NH] nullable
  float* dt_out;       // [n_local x NH] nullable
  float* ds_dir;       // [n_local x NH] directed patterns: row-pass ds for the column pass
  const bf16* P16;     // BF16 mode (reading B1): P and G stored as bfloat16 (P, G unused)
  const bf16* G16;
  const float* ds_row; // [n_local x NH] factored backward: ds_j = G_j . Q_j (prologue)
};

// The factored GAT backward (symmetric patterns; k' = 128 by default, every width
// or none with agnn_plan_options.gat_factored).  With c_ji = alpha_ji lambda_ji (lambda = LReLU slope of the
// entry), the row-role sum of PAPER.md:250-254 is linear in the gathered rows,
//   ds_j = sum_i c_ji (G_j . P_i - delta_j) = G_j . (sum_i c_ji P_i - (sum_i c_ji) Z_j)
//        = G_j . Q_j,
// and the forward already gathers every P_i with its alpha_ji: it accumulates
// Q_j alongside Z_j, the backward prologue forms ds_j = G_j . Q_j, and the
// backward edge pass gathers only G_i and rec_i (column role):
//   dt_j = sum_i c'_ij (G_i . P_j - delta_i) = P_j . v_j - sum_i c'_ij delta_i,
//   v_j = sum_i c'_ij G_i,  acc_j = sum_i alpha_ij G_i.

// k' = 128 kernels (gat_k128.cu): lane-parallel scalar work, warp-parallel rows
bool gat_k128_supported(int k_out, int heads);
agnn_status gat_fwd_k128(const Items& it, int heads, const float* P, const float* st, float slope,
                         int act, const GatFwdOut& o, cudaStream_t s);
// short rows (gat_short.cu): rows of it.short_rows, 4 rows per warp
template <typename TP>
agnn_status gat_fwd_short(const Items& it, int heads, const TP* P, const float* st, float slope,
                          int act, const GatFwdOut& o, cudaStream_t s);
agnn_status gat_bwd_short(const Items& it, int heads, const GatBwdArgs& A, int64_t da_row0,
                          int64_t* warps, cudaStream_t s);
// the k' = 128 row kernels take the long light rows; the short ones go to gat_short.cu
inline Items long_items(const Items& it) {
  Items r = it;
  if (it.n_short > 0) {
    r.light_rows = it.long_rows;
    r.n_light = it.n_long;
  }
  return r;
}
// BF16 mode: P stored as bfloat16
agnn_status gat_fwd_k128_bf16(const Items& it, int heads, const bf16* P, const float* st,
                              float slope, int act, const GatFwdOut& o, cudaStream_t s);
agnn_status gat_bwd_k128(const Items& it, int heads, const GatBwdArgs& A, int64_t* warps,
                         cudaStream_t s);  // A.P16 != NULL: BF16 mode
// factored backward edge pass (A.ds_row set): gathers G_i, rec_i only
agnn_status gat_bwd_k128f(const Items& it, int heads, const GatBwdArgs& A, int64_t* warps,
                          cudaStream_t s);
agnn_status gat_bwd_short_f(const Items& it, int heads, const GatBwdArgs& A, int64_t da_row0,
                            int64_t* warps, cudaStream_t s);
// bundles of short rows (gat_bundle.cu): the short rows as 32-entry warp batches;
// the plan's bundle mode (agnn_plan_options.short_bundles) selects them per storage
// type, else the row-group short kernels (gat_short.cu) run
inline bool gat_bundles_enabled(const Items& it, bool bf16_storage) {
  return bf16_storage ? it.bundle_mode >= 2 : it.bundle_mode >= 1;
}
template <typename TP>
agnn_status gat_fwd_bundle(const Items& it, int heads, const TP* P, const float* st, float slope,
                           int act, const GatFwdOut& o, cudaStream_t s);
agnn_status gat_bwd_bundle(const Items& it, int heads, const GatBwdArgs& A, int64_t da_row0,
                           int64_t* warps, cudaStream_t s);

}  // namespace agnn
