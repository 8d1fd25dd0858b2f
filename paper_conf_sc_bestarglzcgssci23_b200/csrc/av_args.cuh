// av_args.cuh — argument blocks shared by the AGNN / VA sparse kernels
// (agnn_va.cu generic widths, av_batched.cu for k = 128 / 256)
#pragma once
#include "internal.cuh"

namespace agnn {

struct AvFwd {
  const float* H;     // [n_tot x K]  (replicated when world > 1)
  const bf16* H16;    // BF16 mode (reading B2): H~ [n_tot x K] read instead of H
  const float* nu;    // [n_tot]      AGNN
  float beta, bound;  // bound = |beta|
  float* X;           // [n_local x K]
  float* l;           // [n_local]    AGNN
  float* pacc;        // [n_chunks x K]
  float* pl;          // [n_chunks]
};

struct AvBwd {
  const float* H;      // [n_tot x K]
  const float* M;      // [n_tot x K]
  const bf16* H16;     // BF16 mode (reading B2): H~, M~ [n_tot x K] read instead of H, M
  const bf16* M16;
  const float4* rec;   // [n_tot] {nu, m, 1/l, delta}   AGNN
  float beta, eps;
  float* dH;           // [n_local x K]
  float* pacc;         // [n_chunks x 2K]
  float* dhp;          // [n_local x K] directed patterns: row-pass partial of dH (VA) / dH^ (AGNN)
};

enum { AV_VA = 0, AV_AG = 1 };

// k = 128 / 256 batched lane-parallel kernels (av_batched.cu); symmetric patterns
// (ROLE 0) only; AGNN_EUNSUPPORTED for other widths
// (A.H16 != NULL: the BF16 storage variants, same arithmetic on the rounded rows)
agnn_status av_fwd_batched(const Items& it, int k, bool agnn, const AvFwd& A, cudaStream_t s);
// SpMMM, k_in = k_out = 128: X = Psi H and
// Z = X W in one kernel (av_batched.cu), heavy-row chunks and their merge included;
// Z (nullable) and H_out = sigma(Z) are stored by row; store_x: X and l are stored
// too (training: the backward reads them).  hcnt: [n_heavy] ints of workspace.
agnn_status av_fwd_spmmm(const Items& it, bool agnn, const AvFwd& A, const float* W, float* Z,
                         float* H_out, int* hcnt, int act, bool store_x, cudaStream_t s);
agnn_status av_bwd_batched(const Items& it, int k, bool agnn, const AvBwd& A, cudaStream_t s);

}  // namespace agnn
