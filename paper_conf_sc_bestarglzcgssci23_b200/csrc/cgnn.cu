// cgnn.cu — C-GNN layer over a semiring:
//   H_out = sigma((A (x) H) W)            PAPER.md:213 ("C-GNNs ... sigma(A H W)")
// with the aggregation (x) a generalised sparse-dense product over a semiring
// (§4.3): SUM (real semiring), MEAN (averaging semiring),
// GCN (symmetrically normalised A), MAX / MIN (tropical semirings).
//
// Forward: one pass over the CSR (warp per row / heavy-row chunk, lanes own
// 16-byte column slices) producing X (and, for MAX / MIN, the arg index of
// every output element), then Z = X W with sigma in the tcgen05 GEMM epilogue.
// Backward: G = dH_out (.) sigma'(Z); dW = X^T G; M = G W^T (= dL/dX); then
// dH_j = sum over the stored entries (i,j) of coef_ij M_i (SUM / MEAN / GCN) or
// of [arg_ic == j] M_ic (MAX / MIN) — a gather over row j of the symmetric CSR
// (or column j of the plan's CSC for a directed pattern), so no atomics and a
// fixed summation order.
#include "internal.cuh"
#include "warp_batch.cuh"

namespace agnn {
namespace {

constexpr unsigned FULL = 0xffffffffu;

struct CgFwd {
  const float* H;       // [n_tot x K]
  const float* rdeg;    // [n_tot] 1/d (MEAN) or 1/sqrt(d) (GCN)
  float* X;             // [n_local x K]
  int32_t* arg;         // [n_tot x K] (rows at their global offset)  MAX / MIN
  float* pacc;          // [chunks x K]
  int32_t* pidx;        // [chunks x K]  MAX / MIN
};

struct CgBwd {
  const float* M;       // [n_tot x K]
  const float* rdeg;    // [n_tot]
  const int32_t* arg;   // [n_tot x K]
  float* dH;            // [n_local x K]
  float* pacc;          // [chunks x K]
};

__device__ __forceinline__ bool better(int agg, float v, int j, float b, int bj) {
  // strict improvement, ties to the smaller column index (reading C4)
  if (bj < 0) return true;
  if (agg == AGNN_AGG_MAX) return v > b || (v == b && j < bj);
  return v < b || (v == b && j < bj);
}

template <int K, int AGG>
__global__ void __launch_bounds__(kSparseThreads) cg_fwd_kernel(Items it, CgFwd A) {
  using L = RowLayout<K, 1>;
  constexpr bool TROP = AGG == AGNN_AGG_MAX || AGG == AGNN_AGG_MIN;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    wb::item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float acc[L::VPL][4];
    int idx[L::VPL][4];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v)
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        acc[v][x] = 0.f;
        idx[v][x] = -1;
      }
    for (int64_t e = beg + g; e < end; e += L::GROUPS) {
      const int j = __ldg(it.col + e);
      const float cj = (AGG == AGNN_AGG_GCN) ? __ldg(A.rdeg + j) : 1.f;
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        const float4 h = ldg4(A.H + (int64_t)j * K + L::col(v, q));
        const float hv[4] = {h.x, h.y, h.z, h.w};
#pragma unroll
        for (int x = 0; x < 4; ++x) {
          if (TROP) {
            if (better(AGG, hv[x], j, acc[v][x], idx[v][x])) {
              acc[v][x] = hv[x];
              idx[v][x] = j;
            }
          } else {
            acc[v][x] = fmaf(cj, hv[x], acc[v][x]);
          }
        }
      }
    }
    // combine the lane groups (disjoint edge subsets of the row)
#pragma unroll
    for (int off = L::LANES; off < 32; off <<= 1) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v)
#pragma unroll
        for (int x = 0; x < 4; ++x) {
          const float o = __shfl_xor_sync(FULL, acc[v][x], off);
          if (TROP) {
            const int oj = __shfl_xor_sync(FULL, idx[v][x], off);
            if (oj >= 0 && better(AGG, o, oj, acc[v][x], idx[v][x])) {
              acc[v][x] = o;
              idx[v][x] = oj;
            }
          } else {
            acc[v][x] += o;
          }
        }
    }
    if (g != 0) continue;
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const int c = L::col(v, q);
      if (slot >= 0) {
        st4(A.pacc + slot * K + c, make_float4(acc[v][0], acc[v][1], acc[v][2], acc[v][3]));
        if (TROP)
          *reinterpret_cast<int4*>(A.pidx + slot * K + c) =
              make_int4(idx[v][0], idx[v][1], idx[v][2], idx[v][3]);
      } else if (TROP) {
        float4 o;
        o.x = idx[v][0] < 0 ? 0.f : acc[v][0];
        o.y = idx[v][1] < 0 ? 0.f : acc[v][1];
        o.z = idx[v][2] < 0 ? 0.f : acc[v][2];
        o.w = idx[v][3] < 0 ? 0.f : acc[v][3];
        st4(A.X + row * K + c, o);
        *reinterpret_cast<int4*>(A.arg + grow * K + c) =
            make_int4(idx[v][0], idx[v][1], idx[v][2], idx[v][3]);
      } else {
        const float sc = (AGG == AGNN_AGG_SUM) ? 1.f : __ldg(A.rdeg + grow);
        st4(A.X + row * K + c,
            make_float4(sc * acc[v][0], sc * acc[v][1], sc * acc[v][2], sc * acc[v][3]));
      }
    }
  }
}

// heavy rows: fold the chunk partials in ascending chunk order
template <int K, int AGG>
__global__ void __launch_bounds__(kSparseThreads) cg_fwd_merge_kernel(Items it, CgFwd A) {
  using L = RowLayout<K, 1>;
  constexpr bool TROP = AGG == AGNN_AGG_MAX || AGG == AGNN_AGG_MIN;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t h = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; h < it.n_heavy; h += nw) {
    if (g != 0) continue;
    const int64_t row = it.heavy_rows[h], grow = it.row_begin + row;
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const int c = L::col(v, q);
      float a[4] = {0.f, 0.f, 0.f, 0.f};
      int b[4] = {-1, -1, -1, -1};
      for (int64_t s = it.heavy_off[h]; s < it.heavy_off[h + 1]; ++s) {
        const float4 pv = ldg4(A.pacc + s * K + c);
        const float pa[4] = {pv.x, pv.y, pv.z, pv.w};
        if (TROP) {
          const int4 pj = *reinterpret_cast<const int4*>(A.pidx + s * K + c);
          const int pb[4] = {pj.x, pj.y, pj.z, pj.w};
#pragma unroll
          for (int x = 0; x < 4; ++x)
            if (pb[x] >= 0 && better(AGG, pa[x], pb[x], a[x], b[x])) {
              a[x] = pa[x];
              b[x] = pb[x];
            }
        } else {
#pragma unroll
          for (int x = 0; x < 4; ++x) a[x] += pa[x];
        }
      }
      if (TROP) {
        st4(A.X + row * K + c, make_float4(b[0] < 0 ? 0.f : a[0], b[1] < 0 ? 0.f : a[1],
                                           b[2] < 0 ? 0.f : a[2], b[3] < 0 ? 0.f : a[3]));
        *reinterpret_cast<int4*>(A.arg + grow * K + c) = make_int4(b[0], b[1], b[2], b[3]);
      } else {
        const float sc = (AGG == AGNN_AGG_SUM) ? 1.f : __ldg(A.rdeg + grow);
        st4(A.X + row * K + c, make_float4(sc * a[0], sc * a[1], sc * a[2], sc * a[3]));
      }
    }
  }
}

// dH_j = sum over stored (i,j): coef_ij M_i, or [arg_ic == j] M_ic
template <int K, int AGG>
__global__ void __launch_bounds__(kSparseThreads) cg_bwd_kernel(Items it, CgBwd A) {
  using L = RowLayout<K, 1>;
  constexpr bool TROP = AGG == AGNN_AGG_MAX || AGG == AGNN_AGG_MIN;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    wb::item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float4 acc[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) acc[v] = f4(0.f);
    for (int64_t e = beg + g; e < end; e += L::GROUPS) {
      const int i = __ldg(it.col + e);
      const float ci = (AGG == AGNN_AGG_MEAN || AGG == AGNN_AGG_GCN) ? __ldg(A.rdeg + i) : 1.f;
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        const int c = L::col(v, q);
        const float4 m = ldg4(A.M + (int64_t)i * K + c);
        if (TROP) {
          const int4 a = *reinterpret_cast<const int4*>(A.arg + (int64_t)i * K + c);
          acc[v].x += a.x == (int)grow ? m.x : 0.f;
          acc[v].y += a.y == (int)grow ? m.y : 0.f;
          acc[v].z += a.z == (int)grow ? m.z : 0.f;
          acc[v].w += a.w == (int)grow ? m.w : 0.f;
        } else {
          acc[v] = fma4(ci, m, acc[v]);
        }
      }
    }
#pragma unroll
    for (int off = L::LANES; off < 32; off <<= 1)
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        acc[v].x += __shfl_xor_sync(FULL, acc[v].x, off);
        acc[v].y += __shfl_xor_sync(FULL, acc[v].y, off);
        acc[v].z += __shfl_xor_sync(FULL, acc[v].z, off);
        acc[v].w += __shfl_xor_sync(FULL, acc[v].w, off);
      }
    if (g != 0) continue;
    const float sc = (AGG == AGNN_AGG_GCN && slot < 0) ? __ldg(A.rdeg + grow) : 1.f;
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const int c = L::col(v, q);
      if (slot >= 0) st4(A.pacc + slot * K + c, acc[v]);
      else st4(A.dH + row * K + c, mul4(sc, acc[v]));
    }
  }
}

template <int K, int AGG>
__global__ void __launch_bounds__(kSparseThreads) cg_bwd_merge_kernel(Items it, CgBwd A) {
  using L = RowLayout<K, 1>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t h = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; h < it.n_heavy; h += nw) {
    if (g != 0) continue;
    const int64_t row = it.heavy_rows[h], grow = it.row_begin + row;
    const float sc = (AGG == AGNN_AGG_GCN) ? __ldg(A.rdeg + grow) : 1.f;
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const int c = L::col(v, q);
      float4 a = f4(0.f);
      for (int64_t s = it.heavy_off[h]; s < it.heavy_off[h + 1]; ++s)
        a = add4(a, ldg4(A.pacc + s * K + c));
      st4(A.dH + row * K + c, mul4(sc, a));
    }
  }
}

// rdeg_i = 1/d_i (MEAN) or 1/sqrt(d_i) (GCN), d_i = stored entries of row i (0 if empty)
__global__ void cg_rdeg_kernel(const int64_t* __restrict__ rp, int64_t n_local, int64_t row_begin,
                               int agg, float* __restrict__ rdeg) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_local;
       i += (int64_t)gridDim.x * blockDim.x) {
    const float d = (float)(rp[i + 1] - rp[i]);
    rdeg[row_begin + i] = d > 0.f ? (agg == AGNN_AGG_MEAN ? 1.f / d : rsqrtf(d)) : 0.f;
  }
}

__global__ void cg_grad_act_kernel(const float* __restrict__ dHout, const float* __restrict__ Z,
                                   int64_t count4, int act, float* __restrict__ G) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count4;
       i += (int64_t)gridDim.x * blockDim.x) {
    const float4 z = ldg4(Z + 4 * i), d = ldg4(dHout + 4 * i);
    st4(G + 4 * i, make_float4(d.x * act_grad(act, z.x), d.y * act_grad(act, z.y),
                               d.z * act_grad(act, z.z), d.w * act_grad(act, z.w)));
  }
}

// ---------------------------------------------------------------- layout
bool trop(const agnn_layer_desc& d) { return d.agg == AGNN_AGG_MAX || d.agg == AGNN_AGG_MIN; }

struct SavedCg {
  float *Hfull, *X, *Z, *rdeg;
  int32_t* arg;
};
SavedCg carve_saved(const Plan& p, const agnn_layer_desc& d, void* base, size_t* total) {
  Carver c(base);
  SavedCg s;
  // replicated (n-row) arrays first (same offsets on every rank; peer exchange)
  s.Hfull = c.take<float>(p.world > 1 ? (size_t)p.n * d.k_in : 0);
  s.rdeg = c.take<float>((size_t)p.n);
  s.arg = c.take<int32_t>(trop(d) ? (size_t)p.n * d.k_in : 0);
  s.X = c.take<float>((size_t)p.n_local * d.k_in);
  s.Z = c.take<float>((size_t)p.n_local * d.k_out);
  if (total) *total = c.off + 256;
  return s;
}
struct WsCg {
  float *pacc, *G, *M, *gemm, *WT;
  int32_t* pidx;
  void* saved_inf;
};
WsCg carve_ws(const Plan& p, const agnn_layer_desc& d, void* base, size_t* total) {
  Carver c(base);
  WsCg w;
  size_t sv = 0;
  carve_saved(p, d, nullptr, &sv);
  w.M = c.take<float>((size_t)p.n * d.k_in);  // replicated first (peer exchange)
  w.saved_inf = c.take<char>(sv);             // its replicated prefix too
  w.pacc = c.take<float>((size_t)p.max_chunks() * d.k_in);
  w.pidx = c.take<int32_t>(trop(d) ? (size_t)p.max_chunks() * d.k_in : 0);
  w.G = c.take<float>((size_t)p.n_local * d.k_out);
  w.gemm = c.take<float>(gemm_tn_ws_floats(d.k_in, d.k_out));
  w.WT = c.take<float>((size_t)d.k_in * d.k_out);
  if (total) *total = c.off + 256;
  return w;
}

#define AGNN_CG_DISPATCH(K_, AGG_, CALL)                                                  \
  do {                                                                                    \
    bool _done = false;                                                                   \
    AGNN_CG_K(16, K_, AGG_, CALL) AGNN_CG_K(32, K_, AGG_, CALL) AGNN_CG_K(64, K_, AGG_, CALL) \
    AGNN_CG_K(128, K_, AGG_, CALL) AGNN_CG_K(256, K_, AGG_, CALL)                         \
    if (!_done) return fail(AGNN_EUNSUPPORTED, "C-GNN: k_in must be 16/32/64/128/256");   \
  } while (0)
#define AGNN_CG_K(KK, K_, AGG_, CALL)                                                   \
  if (!_done && K_ == KK) {                                                             \
    constexpr int K = KK;                                                               \
    switch (AGG_) {                                                                     \
      case AGNN_AGG_SUM: { constexpr int AGG = AGNN_AGG_SUM; CALL; break; }             \
      case AGNN_AGG_MEAN: { constexpr int AGG = AGNN_AGG_MEAN; CALL; break; }           \
      case AGNN_AGG_GCN: { constexpr int AGG = AGNN_AGG_GCN; CALL; break; }             \
      case AGNN_AGG_MAX: { constexpr int AGG = AGNN_AGG_MAX; CALL; break; }             \
      default: { constexpr int AGG = AGNN_AGG_MIN; CALL; break; }                       \
    }                                                                                   \
    _done = true;                                                                       \
  }

}  // namespace

agnn_status cg_saved_bytes(const Plan& p, const agnn_layer_desc& d, size_t* b) {
  carve_saved(p, d, nullptr, b);
  return AGNN_OK;
}
agnn_status cg_workspace_bytes(const Plan& p, const agnn_layer_desc& d, size_t* b) {
  carve_ws(p, d, nullptr, b);
  return AGNN_OK;
}

agnn_status cg_forward(const Plan& p, const agnn_layer_desc& d, const float* W, const float* H_in,
                       float* H_out, void* saved, void* ws, cudaStream_t s) {
  WsCg w = carve_ws(p, d, ws, nullptr);
  SavedCg sv = carve_saved(p, d, saved ? saved : w.saved_inf, nullptr);
  const int K_ = d.k_in, AGG_ = (int)d.agg;
  agnn_status st;
  const float* Hf = H_in;
  if (p.n_local > 0) {
    cg_rdeg_kernel<<<kNumSMs * 4, 256, 0, s>>>(p.row_ptr, p.n_local, p.row_begin, AGG_, sv.rdeg);
    AGNN_LAUNCH_CHECK("cg_rdeg_kernel");
  }
  if (p.world > 1) {
    AGNN_CUDA_TRY(cudaMemcpyAsync(sv.Hfull + p.row_begin * d.k_in, H_in,
                                  sizeof(float) * p.n_local * d.k_in, cudaMemcpyDeviceToDevice, s));
    const RowArray ra[2] = {{sv.Hfull, d.k_in}, {sv.rdeg, 1}};
    if ((st = allgather_rows(p, ra, 2, s)) != AGNN_OK) return st;
    Hf = sv.Hfull;
  }
  Items it = items_of(p);
  CgFwd A{Hf, sv.rdeg, sv.X, sv.arg, w.pacc, w.pidx};
  if (it.n_chunks + it.n_light > 0) {
    AGNN_CG_DISPATCH(K_, AGG_, (cg_fwd_kernel<K, AGG><<<grid_of(cg_fwd_kernel<K, AGG>),
                                                       kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("cg_fwd_kernel");
  }
  if (it.n_heavy > 0) {
    AGNN_CG_DISPATCH(K_, AGG_, (cg_fwd_merge_kernel<K, AGG><<<kNumSMs * 2, kSparseThreads, 0, s>>>(
                                   it, A)));
    AGNN_LAUNCH_CHECK("cg_fwd_merge_kernel");
  }
  if (p.world > 1 && trop(d))  // the backward gathers the neighbours' arg rows
    if ((st = allgather_rows(p, reinterpret_cast<float*>(sv.arg), d.k_in, s)) != AGNN_OK) return st;
  // Z = X W ; H_out = sigma(Z)   (B = W^T as [k_out x k_in] for the tensor-core path)
  if ((st = transpose(W, d.k_in, d.k_out, w.WT, s)) != AGNN_OK) return st;
  return gemm_rows(sv.X, p.n_local, d.k_in, w.WT, true, d.k_out, saved ? sv.Z : nullptr, d.k_out,
                   nullptr, s, H_out, (int)d.act);
}

agnn_status cg_backward(const Plan& p, const agnn_layer_desc& d, const float* W,
                        const float* H_in, const void* saved, const float* dH_out, float* dH_in,
                        float* dW, void* ws, cudaStream_t s) {
  (void)H_in;
  if (!saved) return fail(AGNN_EINVAL, "agnn_backward: saved == NULL");
  const bool directed = p.directed();
  if (directed && !p.csc_ptr)
    return fail(AGNN_EUNSUPPORTED,
                "agnn_backward: a directed pattern needs world == 1 and every row in the plan");
  WsCg w = carve_ws(p, d, ws, nullptr);
  SavedCg sv = carve_saved(p, d, const_cast<void*>(saved), nullptr);
  const int K_ = d.k_in, AGG_ = (int)d.agg;
  agnn_status st;
  const int64_t c4 = p.n_local * d.k_out / 4;
  if (c4 > 0) {
    cg_grad_act_kernel<<<kNumSMs * 8, kSparseThreads, 0, s>>>(dH_out, sv.Z, c4, (int)d.act, w.G);
    AGNN_LAUNCH_CHECK("grad_act_kernel");
  }
  // Y = dW = X^T G
  if ((st = gemm_tn(sv.X, p.n_local, d.k_in, w.G, d.k_out, dW, w.gemm, s)) != AGNN_OK) return st;
  if (p.world > 1 && (st = allreduce_sum(p, dW, (int64_t)d.k_in * d.k_out, s)) != AGNN_OK) return st;
  if (!dH_in) return AGNN_OK;
  // M = G W^T = dL/dX
  if ((st = gemm_rows(w.G, p.n_local, d.k_out, W, true, d.k_in, w.M + p.row_begin * d.k_in, d.k_in,
                      nullptr, s)) != AGNN_OK)
    return st;
  if (p.world > 1 && (st = allgather_rows(p, w.M, d.k_in, s)) != AGNN_OK) return st;
  // dH_j gathers over the entries (i,j): row j of the symmetric CSR, or column j of the CSC
  Items it = directed ? items_of_csc(p) : items_of(p);
  CgBwd A{w.M, sv.rdeg, sv.arg, dH_in, w.pacc};
  if (it.n_chunks + it.n_light > 0) {
    AGNN_CG_DISPATCH(K_, AGG_, (cg_bwd_kernel<K, AGG><<<grid_of(cg_bwd_kernel<K, AGG>),
                                                       kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("cg_bwd_kernel");
  }
  if (it.n_heavy > 0) {
    AGNN_CG_DISPATCH(K_, AGG_, (cg_bwd_merge_kernel<K, AGG><<<kNumSMs * 2, kSparseThreads, 0, s>>>(
                                   it, A)));
    AGNN_LAUNCH_CHECK("cg_bwd_merge_kernel");
  }
  return AGNN_OK;
}

}  // namespace agnn
