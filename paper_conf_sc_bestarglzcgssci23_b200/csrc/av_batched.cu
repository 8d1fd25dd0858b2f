// av_batched.cu — AGNN / VA sparse kernels for k = 128 and 256 (the C3 and C4
// shapes), organised like gat_k128.cu: feature-row work warp-parallel (lane q
// owns columns 4q..4q+3 of every 128-column block), scalar per-edge work
// lane-parallel.
//
// Arithmetic is exactly that of agnn_va.cu (PAPER.md:173/:175 scores, Eq. 7;
// PAPER.md:250-254 backward, VA Eq. 11-13; reading A8: softmax with the fixed
// shift |beta|, so the weights need no running max).  What changes is the
// reduction: the generic kernels reduce every per-edge dot product over the 32
// lanes separately (5 shuffles per dot, 3 dots per edge in the backward).  Here
// a batch of B edges is gathered, each lane forms its B partial dots, and the
// transposed butterfly (warp_batch.cuh) leaves lane b with the full dots of
// edge b in log2(B) + (5 - log2 B) steps for all B at once; the lane computes
// that edge's coefficients and they are broadcast back for the row updates.
#include "av_args.cuh"
#include "warp_batch.cuh"

namespace agnn {
namespace {

using wb::FULL;
using wb::item_of;
using wb::Transpose;

// TP = float (fp32 rows) or bf16 (BF16 storage, reading B2): the batches hold the raw
// loaded slices and widen them at use, so a batch's loads stay in flight while the
// previous batch is computed
template <int B, int V, typename TP>
struct FwdBatch {
  typename Slice<TP>::raw Hj[B][V];
  float nuj;  // nu of the edge this lane owns after the reduction (AGNN)
};
template <typename TP>
__device__ __forceinline__ const TP* pick_row(const float* f, const bf16* h);
template <>
__device__ __forceinline__ const float* pick_row<float>(const float* f, const bf16*) { return f; }
template <>
__device__ __forceinline__ const bf16* pick_row<bf16>(const float*, const bf16* h) { return h; }

template <int V>
__device__ __forceinline__ float dotv(const float4 (&a)[V], const float4 (&b)[V]) {
  float d = dot4(a[0], b[0]);
#pragma unroll
  for (int v = 1; v < V; ++v) d += dot4(a[v], b[v]);
  return d;
}

// X_i = sum_j w_ij H_j, w = exp(beta cos(H_i, H_j) - |beta|) (AGNN, l_i = sum w) or
// w = H_i . H_j (VA)
template <int K, int MODEL, int B, int MINB, typename TP>
__global__ void __launch_bounds__(256, MINB) av_fwd_batched_kernel(Items it, AvFwd A) {
  constexpr int V = K / 128;
  using TR = Transpose<B>;
  using SL = Slice<TP>;
  const TP* Hrow = pick_row<TP>(A.H, A.H16);
  const int lane = threadIdx.x & 31, cq = lane * 4;
  const int my_b = TR::edge_of(lane);
  const bool owner = (lane >> TR::T) == 0;
  const float beta = A.beta, bound = A.bound;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const TP* Hl = Hrow + cq;
  const Gath ga(it);  // L2 residency hints of the gathered rows (plan column classes)
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float4 Hi[V], acc[V];
#pragma unroll
    for (int v = 0; v < V; ++v) {
      Hi[v] = SL::f(SL::load(Hrow + grow * K + v * 128 + cq));
      acc[v] = f4(0.f);
    }
    const float scale_i = (MODEL == AV_AG) ? beta / __ldg(A.nu + grow) : 1.f;
    float lp = 0.f;
    auto load = [&](FwdBatch<B, V, TP>& q, int cidx, int off, int cnt) {
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const int c = __shfl_sync(FULL, cidx, off + b);
        const int64_t j = ga.row(c);
        const uint64_t pol = ga.policy(c);
#pragma unroll
        for (int v = 0; v < V; ++v)
          q.Hj[b][v] = b < cnt ? SL::load(Hl + j * K + v * 128, pol) : SL::zero();
      }
      if (MODEL == AV_AG) {
        const int cm = __shfl_sync(FULL, cidx, off + my_b);
        q.nuj = my_b < cnt ? ldg1_pol(A.nu + ga.row(cm), ga.policy(cm)) : 1.f;
      }
    };
    auto body = [&](const FwdBatch<B, V, TP>& q, int cnt) {
      float4 Hj[B][V];
#pragma unroll
      for (int b = 0; b < B; ++b)
#pragma unroll
        for (int v = 0; v < V; ++v) Hj[b][v] = SL::f(q.Hj[b][v]);
      float x[B];
#pragma unroll
      for (int b = 0; b < B; ++b) x[b] = dotv<V>(Hi, Hj[b]);
      TR::template reduce<32>(x, lane);
      float wgt;
      if (MODEL == AV_AG) wgt = ex2((scale_i * x[0] / q.nuj - bound) * kLog2e);  // exp(c_ij - |beta|)
      else wgt = x[0];                                                           // S_ij = H_i . H_j
      if (my_b >= cnt) wgt = 0.f;
      if (MODEL == AV_AG && owner) lp += wgt;
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const float wbv = __shfl_sync(FULL, wgt, TR::lane_of(b));
#pragma unroll
        for (int v = 0; v < V; ++v) acc[v] = fma4(wbv, Hj[b][v], acc[v]);
      }
    };
    for (int64_t w0 = beg; w0 < end; w0 += 32) {
      const int wcnt = (int)(end - w0 < 32 ? end - w0 : 32);
      const int cidx = lane < wcnt ? __ldg(it.col + w0 + lane) : 0;
      if (wcnt == 32) {
        FwdBatch<B, V, TP> qa, qb;
        load(qa, cidx, 0, B);
#pragma unroll
        for (int bb = 0; bb < 32 / B; bb += 2) {
          load(qb, cidx, (bb + 1) * B, B);
          body(qa, B);
          if (bb + 2 < 32 / B) load(qa, cidx, (bb + 2) * B, B);
          body(qb, B);
        }
      } else {
        for (int off = 0; off < wcnt; off += B) {
          FwdBatch<B, V, TP> q;
          const int cnt = wcnt - off < B ? wcnt - off : B;
          load(q, cidx, off, cnt);
          body(q, cnt);
        }
      }
    }
    float l = 0.f;
    if (MODEL == AV_AG) {
      l = lp;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) l += __shfl_xor_sync(FULL, l, o);
    }
    if (slot >= 0) {
#pragma unroll
      for (int v = 0; v < V; ++v) st4(A.pacc + slot * K + v * 128 + cq, acc[v]);
      if (MODEL == AV_AG && lane == 0) A.pl[slot] = l;
    } else {
      const float inv = (MODEL == AV_AG) ? (l > 0.f ? 1.f / l : 0.f) : 1.f;
#pragma unroll
      for (int v = 0; v < V; ++v) st4(A.X + row * K + v * 128 + cq, mul4(inv, acc[v]));
      if (MODEL == AV_AG && lane == 0) A.l[row] = l;
    }
  }
}

template <int B, int V, typename TP>
struct BwdBatchAV {
  typename Slice<TP>::raw Hi[B][V], Mi[B][V];
  float4 ri;  // record {nu, m, 1/l, delta} of the owned edge's vertex (AGNN)
};

// One pass over the symmetric CSR, both roles of every stored entry (j,i):
//   VA   dH_j += (M_j.H_i + M_i.H_j) H_i + (H_i.H_j) M_i
//   AGNN dH^_j += beta (a_ji (M_j.H_i - d_j) + a_ij (M_i.H_j - d_i)) H^_i,
//        acc_j += a_ij M_i ;  dH_j = acc_j + (dH^_j - (dH^_j.H^_j) H^_j) / nu_j
template <int K, int MODEL, int B, int MINB, typename TP>
__global__ void __launch_bounds__(256, MINB) av_bwd_batched_kernel(Items it, AvBwd A) {
  constexpr int V = K / 128;
  using TR = Transpose<B>;
  using SL = Slice<TP>;
  const TP* Hrow = pick_row<TP>(A.H, A.H16);
  const TP* Mrow = pick_row<TP>(A.M, A.M16);
  const int lane = threadIdx.x & 31, cq = lane * 4;
  const int my_b = TR::edge_of(lane);
  const float beta = A.beta;
  const int64_t nitems = it.n_chunks + it.n_light;
  const Gath ga(it);
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const TP* Hl = Hrow + cq;
  const TP* Ml = Mrow + cq;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float4 Hj[V], Mj[V], dh[V], acc[V];
#pragma unroll
    for (int v = 0; v < V; ++v) {
      Hj[v] = SL::f(SL::load(Hrow + grow * K + v * 128 + cq));
      Mj[v] = SL::f(SL::load(Mrow + grow * K + v * 128 + cq));
      dh[v] = acc[v] = f4(0.f);
    }
    const float4 rj = (MODEL == AV_AG) ? __ldg(A.rec + grow) : f4(1.f);
    const float sj = (MODEL == AV_AG) ? beta / rj.x : 0.f;
    auto load = [&](BwdBatchAV<B, V, TP>& q, int cidx, int off, int cnt) {
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const int c = __shfl_sync(FULL, cidx, off + b);
        const int64_t i = ga.row(c);
        const uint64_t pol = ga.policy(c);
#pragma unroll
        for (int v = 0; v < V; ++v) {
          if (b < cnt) {
            q.Hi[b][v] = SL::load(Hl + i * K + v * 128, pol);
            q.Mi[b][v] = SL::load(Ml + i * K + v * 128, pol);
          } else {
            q.Hi[b][v] = q.Mi[b][v] = SL::zero();
          }
        }
      }
      if (MODEL == AV_AG) {
        const int cm = __shfl_sync(FULL, cidx, off + my_b);
        q.ri = my_b < cnt ? ldg4_pol(reinterpret_cast<const float*>(A.rec + ga.row(cm)), ga.policy(cm))
                          : f4(1.f);
      }
    };
    auto body = [&](const BwdBatchAV<B, V, TP>& q, int cnt) {
      float4 Hi[B][V], Mi[B][V];
#pragma unroll
      for (int b = 0; b < B; ++b)
#pragma unroll
        for (int v = 0; v < V; ++v) {
          Hi[b][v] = SL::f(q.Hi[b][v]);
          Mi[b][v] = SL::f(q.Mi[b][v]);
        }
      float xs[B], x1[B], x2[B];
#pragma unroll
      for (int b = 0; b < B; ++b) {
        xs[b] = dotv<V>(Hj, Hi[b]);   // H_j . H_i
        x1[b] = dotv<V>(Mj, Hi[b]);   // M_j . H_i  (row role)
        x2[b] = dotv<V>(Mi[b], Hj);   // M_i . H_j  (column role)
      }
      TR::template reduce<32>(xs, lane);
      TR::template reduce<32>(x1, lane);
      TR::template reduce<32>(x2, lane);
      float ch, cm;  // coefficients of H_i and M_i for the owned edge
      if (MODEL == AV_VA) {
        ch = x1[0] + x2[0];
        cm = xs[0];
      } else {
        const float inv_nui = 1.f / q.ri.x;
        const float c = sj * xs[0] * inv_nui;                       // beta cos(H_j, H_i)
        const float aji = ex2((c - rj.y) * kLog2e) * rj.z;          // alpha_ji (row j)
        const float aij = ex2((c - q.ri.y) * kLog2e) * q.ri.z;      // alpha_ij (row i)
        const float dc = beta * (aji * (x1[0] - rj.w) + aij * (x2[0] - q.ri.w));
        ch = dc * inv_nui;                                          // dH^_j += dc H^_i
        cm = aij;                                                   // acc_j += alpha_ij M_i
      }
      if (my_b >= cnt) ch = cm = 0.f;
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const float chb = __shfl_sync(FULL, ch, TR::lane_of(b));
        const float cmb = __shfl_sync(FULL, cm, TR::lane_of(b));
#pragma unroll
        for (int v = 0; v < V; ++v) {
          dh[v] = fma4(chb, Hi[b][v], dh[v]);
          if (MODEL == AV_VA) dh[v] = fma4(cmb, Mi[b][v], dh[v]);
          else acc[v] = fma4(cmb, Mi[b][v], acc[v]);
        }
      }
    };
    for (int64_t w0 = beg; w0 < end; w0 += 32) {
      const int wcnt = (int)(end - w0 < 32 ? end - w0 : 32);
      const int cidx = lane < wcnt ? __ldg(it.col + w0 + lane) : 0;
      if (wcnt == 32) {
        BwdBatchAV<B, V, TP> qa, qb;
        load(qa, cidx, 0, B);
#pragma unroll
        for (int bb = 0; bb < 32 / B; bb += 2) {
          load(qb, cidx, (bb + 1) * B, B);
          body(qa, B);
          if (bb + 2 < 32 / B) load(qa, cidx, (bb + 2) * B, B);
          body(qb, B);
        }
      } else {
        for (int off = 0; off < wcnt; off += B) {
          BwdBatchAV<B, V, TP> q;
          const int cnt = wcnt - off < B ? wcnt - off : B;
          load(q, cidx, off, cnt);
          body(q, cnt);
        }
      }
    }
    if (slot >= 0) {
#pragma unroll
      for (int v = 0; v < V; ++v) {
        st4(A.pacc + slot * 2 * K + v * 128 + cq, dh[v]);
        if (MODEL == AV_AG) st4(A.pacc + slot * 2 * K + K + v * 128 + cq, acc[v]);
      }
      continue;
    }
    if (MODEL == AV_VA) {
#pragma unroll
      for (int v = 0; v < V; ++v) st4(A.dH + row * K + v * 128 + cq, dh[v]);
    } else {
      // dH_j = acc_j + (dH^_j - (dH^_j . H^_j) H^_j) / nu_j   (nu const on the eps branch)
      float pr = dotv<V>(dh, Hj);
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) pr += __shfl_xor_sync(FULL, pr, o);
      const float nuj = rj.x;
      const bool on_eps = !(nuj > A.eps);
      const float inv = 1.f / nuj;
      const float proj = on_eps ? 0.f : pr * inv * inv;
#pragma unroll
      for (int v = 0; v < V; ++v) {
        float4 gv = fma4(-proj, Hj[v], dh[v]);
        gv = fma4(inv, gv, acc[v]);
        st4(A.dH + row * K + v * 128 + cq, gv);
      }
    }
  }
}

template <typename F>
int grid_for(F* f) {
  return persistent_blocks(reinterpret_cast<const void*>(f));
}

// batch sizes / residency measured at C3 (AGNN, R-MAT 2^20, k = 128): forward B = 8,
// backward B = 4 (two batches of H_i, M_i in flight), 2 CTAs of 256 per SM; larger
// batches or 3 CTAs per SM spill and lose 10-40 %.  k = 256 halves the batches
// (same registers per batch).
// (BF16 storage keeps the same batches: half the bytes per gathered row)
template <int K, int MODEL>
void launch_fwd(const Items& it, const AvFwd& A, cudaStream_t s) {
  if (A.H16) {
    auto k = av_fwd_batched_kernel<K, MODEL, K == 128 ? 8 : 4, 2, bf16>;
    k<<<grid_for(k), 256, 0, s>>>(it, A);
  } else {
    auto k = av_fwd_batched_kernel<K, MODEL, K == 128 ? 8 : 4, 2, float>;
    k<<<grid_for(k), 256, 0, s>>>(it, A);
  }
}
template <int K, int MODEL>
void launch_bwd(const Items& it, const AvBwd& A, cudaStream_t s) {
  if (A.H16) {
    auto k = av_bwd_batched_kernel<K, MODEL, K == 128 ? 4 : 2, 2, bf16>;
    k<<<grid_for(k), 256, 0, s>>>(it, A);
  } else {
    auto k = av_bwd_batched_kernel<K, MODEL, K == 128 ? 4 : 2, 2, float>;
    k<<<grid_for(k), 256, 0, s>>>(it, A);
  }
}

}  // namespace

agnn_status av_fwd_batched(const Items& it, int k, bool agnn, const AvFwd& A, cudaStream_t s) {
  if (it.n_chunks + it.n_light == 0) return AGNN_OK;
  if (k == 128) {
    if (agnn) launch_fwd<128, AV_AG>(it, A, s);
    else launch_fwd<128, AV_VA>(it, A, s);
  } else if (k == 256) {
    if (agnn) launch_fwd<256, AV_AG>(it, A, s);
    else launch_fwd<256, AV_VA>(it, A, s);
  } else {
    return AGNN_EUNSUPPORTED;
  }
  AGNN_LAUNCH_CHECK("av_fwd_kernel");
  return AGNN_OK;
}

agnn_status av_bwd_batched(const Items& it, int k, bool agnn, const AvBwd& A, cudaStream_t s) {
  if (it.n_chunks + it.n_light == 0) return AGNN_OK;
  if (k == 128) {
    if (agnn) launch_bwd<128, AV_AG>(it, A, s);
    else launch_bwd<128, AV_VA>(it, A, s);
  } else if (k == 256) {
    if (agnn) launch_bwd<256, AV_AG>(it, A, s);
    else launch_bwd<256, AV_VA>(it, A, s);
  } else {
    return AGNN_EUNSUPPORTED;
  }
  AGNN_LAUNCH_CHECK("av_bwd_kernel");
  return AGNN_OK;
}

}  // namespace agnn
