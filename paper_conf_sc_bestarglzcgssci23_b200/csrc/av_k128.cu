// av_k128.cu — AGNN / VA sparse kernels for k = 128 (the C3 shape), organised
// like gat_k128.cu: feature-row work warp-parallel (lane q owns columns
// 4q..4q+3), scalar per-edge work lane-parallel.
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

constexpr int K = 128;

template <int B>
struct FwdBatch {
  float4 Hj[B];
  float nuj;  // nu of the edge this lane owns after the reduction (AGNN)
};

// X_i = sum_j w_ij H_j, w = exp(beta cos(H_i, H_j) - |beta|) (AGNN, l_i = sum w) or
// w = H_i . H_j (VA)
template <int MODEL, int B, int MINB>
__global__ void __launch_bounds__(256, MINB) av_fwd_k128_kernel(Items it, AvFwd A) {
  using TR = Transpose<B>;
  const int lane = threadIdx.x & 31, cq = lane * 4;
  const int my_b = TR::edge_of(lane);
  const bool owner = (lane >> TR::T) == 0;
  const float beta = A.beta, bound = A.bound;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const float* Hl = A.H + cq;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    const float4 Hi = ldg4(A.H + grow * K + cq);
    const float scale_i = (MODEL == AV_AG) ? beta / __ldg(A.nu + grow) : 1.f;
    float4 acc = f4(0.f);
    float lp = 0.f;
    auto load = [&](FwdBatch<B>& q, int cidx, int off, int cnt) {
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const uint32_t j = (uint32_t)__shfl_sync(FULL, cidx, off + b);
        q.Hj[b] = b < cnt ? ldg4(Hl + (int64_t)j * K) : f4(0.f);
      }
      if (MODEL == AV_AG) {
        const uint32_t jm = (uint32_t)__shfl_sync(FULL, cidx, off + my_b);
        q.nuj = my_b < cnt ? __ldg(A.nu + jm) : 1.f;
      }
    };
    auto body = [&](const FwdBatch<B>& q, int cnt) {
      float x[B];
#pragma unroll
      for (int b = 0; b < B; ++b) x[b] = dot4(Hi, q.Hj[b]);
      TR::template reduce<32>(x, lane);
      float wgt;
      if (MODEL == AV_AG) wgt = ex2((scale_i * x[0] / q.nuj - bound) * kLog2e);  // exp(c_ij - |beta|)
      else wgt = x[0];                                                           // S_ij = H_i . H_j
      if (my_b >= cnt) wgt = 0.f;
      if (MODEL == AV_AG && owner) lp += wgt;
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const float wbv = __shfl_sync(FULL, wgt, TR::lane_of(b));
        acc = fma4(wbv, q.Hj[b], acc);
      }
    };
    for (int64_t w0 = beg; w0 < end; w0 += 32) {
      const int wcnt = (int)(end - w0 < 32 ? end - w0 : 32);
      const int cidx = lane < wcnt ? __ldg(it.col + w0 + lane) : 0;
      if (wcnt == 32) {
        FwdBatch<B> qa, qb;
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
          FwdBatch<B> q;
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
      st4(A.pacc + slot * K + cq, acc);
      if (MODEL == AV_AG && lane == 0) A.pl[slot] = l;
    } else {
      const float inv = (MODEL == AV_AG) ? (l > 0.f ? 1.f / l : 0.f) : 1.f;
      st4(A.X + row * K + cq, mul4(inv, acc));
      if (MODEL == AV_AG && lane == 0) A.l[row] = l;
    }
  }
}

template <int B>
struct BwdBatchAV {
  float4 Hi[B], Mi[B];
  float4 ri;  // record {nu, m, 1/l, delta} of the owned edge's vertex (AGNN)
};

// One pass over the symmetric CSR, both roles of every stored entry (j,i):
//   VA   dH_j += (M_j.H_i + M_i.H_j) H_i + (H_i.H_j) M_i
//   AGNN dH^_j += beta (a_ji (M_j.H_i - d_j) + a_ij (M_i.H_j - d_i)) H^_i,
//        acc_j += a_ij M_i ;  dH_j = acc_j + (dH^_j - (dH^_j.H^_j) H^_j) / nu_j
template <int MODEL, int B, int MINB>
__global__ void __launch_bounds__(256, MINB) av_bwd_k128_kernel(Items it, AvBwd A) {
  using TR = Transpose<B>;
  const int lane = threadIdx.x & 31, cq = lane * 4;
  const int my_b = TR::edge_of(lane);
  const float beta = A.beta;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const float* Hl = A.H + cq;
  const float* Ml = A.M + cq;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    const float4 Hj = ldg4(A.H + grow * K + cq);
    const float4 Mj = ldg4(A.M + grow * K + cq);
    const float4 rj = (MODEL == AV_AG) ? __ldg(A.rec + grow) : f4(1.f);
    const float sj = (MODEL == AV_AG) ? beta / rj.x : 0.f;
    float4 dh = f4(0.f), acc = f4(0.f);
    auto load = [&](BwdBatchAV<B>& q, int cidx, int off, int cnt) {
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const uint32_t i = (uint32_t)__shfl_sync(FULL, cidx, off + b);
        if (b < cnt) {
          q.Hi[b] = ldg4(Hl + (int64_t)i * K);
          q.Mi[b] = ldg4(Ml + (int64_t)i * K);
        } else {
          q.Hi[b] = q.Mi[b] = f4(0.f);
        }
      }
      if (MODEL == AV_AG) {
        const uint32_t im = (uint32_t)__shfl_sync(FULL, cidx, off + my_b);
        q.ri = my_b < cnt ? __ldg(A.rec + im) : f4(1.f);
      }
    };
    auto body = [&](const BwdBatchAV<B>& q, int cnt) {
      float xs[B], x1[B], x2[B];
#pragma unroll
      for (int b = 0; b < B; ++b) {
        xs[b] = dot4(Hj, q.Hi[b]);   // H_j . H_i
        x1[b] = dot4(Mj, q.Hi[b]);   // M_j . H_i  (row role)
        x2[b] = dot4(q.Mi[b], Hj);   // M_i . H_j  (column role)
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
        dh = fma4(chb, q.Hi[b], dh);
        if (MODEL == AV_VA) dh = fma4(cmb, q.Mi[b], dh);
        else acc = fma4(cmb, q.Mi[b], acc);
      }
    };
    for (int64_t w0 = beg; w0 < end; w0 += 32) {
      const int wcnt = (int)(end - w0 < 32 ? end - w0 : 32);
      const int cidx = lane < wcnt ? __ldg(it.col + w0 + lane) : 0;
      if (wcnt == 32) {
        BwdBatchAV<B> qa, qb;
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
          BwdBatchAV<B> q;
          const int cnt = wcnt - off < B ? wcnt - off : B;
          load(q, cidx, off, cnt);
          body(q, cnt);
        }
      }
    }
    if (slot >= 0) {
      st4(A.pacc + slot * 2 * K + cq, dh);
      if (MODEL == AV_AG) st4(A.pacc + slot * 2 * K + K + cq, acc);
      continue;
    }
    if (MODEL == AV_VA) {
      st4(A.dH + row * K + cq, dh);
    } else {
      // dH_j = acc_j + (dH^_j - (dH^_j . H^_j) H^_j) / nu_j   (nu const on the eps branch)
      float pr = dot4(dh, Hj);
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) pr += __shfl_xor_sync(FULL, pr, o);
      const float nuj = rj.x;
      const bool on_eps = !(nuj > A.eps);
      const float inv = 1.f / nuj;
      const float proj = on_eps ? 0.f : pr * inv * inv;
      float4 gv = fma4(-proj, Hj, dh);
      gv = fma4(inv, gv, acc);
      st4(A.dH + row * K + cq, gv);
    }
  }
}

template <typename F>
int grid_for(F* f) {
  return persistent_blocks(reinterpret_cast<const void*>(f));
}

// batch sizes / residency measured at C3 (AGNN, R-MAT 2^20, k = 128): forward B = 8,
// backward B = 4 (two batches of H_i, M_i in flight), 2 CTAs of 256 per SM; larger
// batches or 3 CTAs per SM spill and lose 10-40 %
template <int MODEL>
void launch_fwd(const Items& it, const AvFwd& A, cudaStream_t s) {
  auto k = av_fwd_k128_kernel<MODEL, 8, 2>;
  k<<<grid_for(k), 256, 0, s>>>(it, A);
}
template <int MODEL>
void launch_bwd(const Items& it, const AvBwd& A, cudaStream_t s) {
  auto k = av_bwd_k128_kernel<MODEL, 4, 2>;
  k<<<grid_for(k), 256, 0, s>>>(it, A);
}

}  // namespace

agnn_status av_fwd_k128(const Items& it, bool agnn, const AvFwd& A, cudaStream_t s) {
  if (it.n_chunks + it.n_light == 0) return AGNN_OK;
  if (agnn) launch_fwd<AV_AG>(it, A, s);
  else launch_fwd<AV_VA>(it, A, s);
  AGNN_LAUNCH_CHECK("av_fwd_kernel");
  return AGNN_OK;
}

agnn_status av_bwd_k128(const Items& it, bool agnn, const AvBwd& A, cudaStream_t s) {
  if (it.n_chunks + it.n_light == 0) return AGNN_OK;
  if (agnn) launch_bwd<AV_AG>(it, A, s);
  else launch_bwd<AV_VA>(it, A, s);
  AGNN_LAUNCH_CHECK("av_bwd_kernel");
  return AGNN_OK;
}

}  // namespace agnn
