// gat_k128.cu — GAT sparse kernels for k' = 128 (the C5 shape), organised so that
// scalar per-edge work runs lane-parallel and only the feature-row work runs
// warp-parallel.
//
// Arithmetic is exactly that of gat.cu (PAPER.md:177 forward with the graph
// softmax of PAPER.md:191; PAPER.md:250-254 backward with Psi^T, readings
// A11/A12), in log2 units (scores s, t and row maxima m pre-scaled by log2 e).
//
// Forward, per row i, edges in batches of 32 (one edge per lane):
//   lane e: t_j (all heads), e_ij = LReLU(s_i + t_j), batch max per head by a
//   warp max; running max / rescale once per batch; p_ij = 2^(e_ij - m).
//   Then the warp walks the batch: lane q owns columns 4q..4q+3 of P_j and
//   accumulates p_ij(head(q)) P_j.  Per edge: one 16-byte gather and 4 FMAs.
//   BF16 storage (256-byte rows): the half-warps take the even / odd entries, two
//   rows per 16-byte-per-lane load instruction (gat_fwd_k128_pair_kernel, and
//   gat_bwd_k128f_pair_kernel for the factored backward).
// Factored backward (default, gat_args.cuh): the forward also accumulates Q_j, and
//   the backward row kernel (gat_bwd_k128f_kernel) keeps only the column role —
//   32-entry windows, lane-parallel alpha_ij / c'_ij from the gathered records,
//   then warp-parallel acc += alpha G_i, v += c' G_i; no per-edge dot products.
// Unfactored backward (AGNN_GAT_FACTORED=0), per row j, edges in batches of B (<= lanes per head):
//   warp-parallel: gather P_i, G_i slices; partial dots G_j.P_i and G_i.P_j;
//   a transposed butterfly reduction leaves each lane with both full dots of
//   ONE edge of its head; lane-parallel scalar work (the two alpha recomputes,
//   dc_ji, dc_ij); alpha_ij is broadcast back for acc_j += alpha_ij G_i.
#include "gat_args.cuh"
#include "warp_batch.cuh"

namespace agnn {
namespace {

using wb::item_of;
using wb::Transpose;

constexpr unsigned FULL = 0xffffffffu;
constexpr int K = 128;

template <int N>
__device__ __forceinline__ void load_n(const float* p, float (&x)[N]) {
  if constexpr (N % 4 == 0) {
#pragma unroll
    for (int i = 0; i < N; i += 4) {
      const float4 v = ldg4(p + i);
      x[i] = v.x;
      x[i + 1] = v.y;
      x[i + 2] = v.z;
      x[i + 3] = v.w;
    }
  } else if constexpr (N == 2) {
    const float2 v = __ldg(reinterpret_cast<const float2*>(p));
    x[0] = v.x;
    x[1] = v.y;
  } else {
#pragma unroll
    for (int i = 0; i < N; ++i) x[i] = __ldg(p + i);
  }
}

// the same with an explicit L2 policy (gathered rows of other vertices)
template <int N>
__device__ __forceinline__ void load_n(const float* p, float (&x)[N], uint64_t pol) {
  if constexpr (N % 4 == 0) {
#pragma unroll
    for (int i = 0; i < N; i += 4) {
      const float4 v = ldg4_pol(p + i, pol);
      x[i] = v.x;
      x[i + 1] = v.y;
      x[i + 2] = v.z;
      x[i + 3] = v.w;
    }
  } else if constexpr (N == 2) {
    const uint2 v = ldg8_pol(p, pol);
    x[0] = __uint_as_float(v.x);
    x[1] = __uint_as_float(v.y);
  } else {
#pragma unroll
    for (int i = 0; i < N; ++i) x[i] = ldg1_pol(p + i, pol);
  }
}

// fp32 rows, or bfloat16 rows (BF16 mode, reading B1): same code, the gathers
// widen 4 bf16 (8 bytes) to a float4 (common.cuh ldg4 overloads)
template <typename TP>
__device__ __forceinline__ const TP* pick(const float* f, const bf16* h);
template <>
__device__ __forceinline__ const float* pick<float>(const float* f, const bf16*) { return f; }
template <>
__device__ __forceinline__ const bf16* pick<bf16>(const float*, const bf16* h) { return h; }

// ---------------------------------------------------------------- forward
// rows per gather group of the full-batch path: 4 fp32 rows (2 KB) or 8 bf16 rows
// (2 KB) per lane-slice group, two groups in flight
template <typename TP>
constexpr int fwd_group() { return sizeof(TP) == 2 ? 8 : 4; }

// QF (training, factored backward): also accumulate u_i = sum_j p_ij lambda_ij P_j and
// C_i = sum_j p_ij lambda_ij with the same online rescaling, and store
// Q_i = (u_i - (C_i / l_i) acc_i) / l_i  (= sum_j c_ij P_j - (sum_j c_ij) Z_i, gat_args.cuh);
// when every lambda_ij = 1 (all pre-activations > 0) u = acc and C = l bitwise, so
// Q = 0 and ds = 0 exactly, as in exact arithmetic.
template <typename TP, int NH, int U, int MINB, bool QF, int GRT = 0>
__global__ void __launch_bounds__(256, MINB)
gat_fwd_k128_kernel(Items it, const TP* __restrict__ P, const float* __restrict__ st,
                    float slope, int act, GatFwdOut o) {
  constexpr int D = K / NH, HL = D / 4;
  // +1: heads read different rows without bank conflicts; QF: {p, p lambda} pairs
  __shared__ float sPw[QF ? 1 : 8][NH][33];
  __shared__ float2 sP2[QF ? 8 : 1][NH][33];
  __shared__ int sJ[8][32];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int hv = lane / HL, cq = lane * 4;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const Gath ga(it);
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float si[NH], mr[NH], lp[NH], lc[NH];
    load_n<NH>(st + grow * (2 * NH), si);
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      mr[h] = -INFINITY;
      lp[h] = 0.f;
      lc[h] = 0.f;
    }
    float4 acc = f4(0.f), accu = f4(0.f);
    // column ids one batch ahead: the next batch's ids load during this batch
    int jpre = beg + lane < end ? __ldg(it.col + beg + lane) : 0;
    for (int64_t b0 = beg; b0 < end; b0 += 32) {
      const int cnt = (int)(end - b0 < 32 ? end - b0 : 32);
      const bool valid = lane < cnt;
      const int j = jpre;
      jpre = b0 + 32 + lane < end ? __ldg(it.col + b0 + 32 + lane) : 0;
      sJ[wib][lane] = j;
      __syncwarp();
      // the first U neighbour rows are in flight while the scores are computed
      using SL = Slice<TP>;
      typename SL::raw pv[U];
#pragma unroll
      for (int u = 0; u < U; ++u)
        pv[u] = u < cnt ? SL::load(P + ga.row(sJ[wib][u]) * K + cq, ga.policy(sJ[wib][u]))
                        : SL::zero();
      float tj[NH];
      load_n<NH>(st + ga.row(j) * (2 * NH) + NH, tj, ga.policy(j));
      float sch = 1.f;
#pragma unroll
      for (int h = 0; h < NH; ++h) {
        const float pre = si[h] + tj[h];
        const float e = valid ? fmaxf(pre, slope * pre) : -INFINITY;  // LReLU, 0 <= slope <= 1
        float bm = e;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) bm = fmaxf(bm, __shfl_xor_sync(FULL, bm, off));
        const float mn = fmaxf(mr[h], bm);
        const float sc = ex2(mr[h] - mn);  // 0 on the first batch (mr = -inf)
        // rounded multiply then add, never contracted: the training (QF) and inference
        // variants must produce bitwise the same l, and lc the same ops as lp
        lp[h] = __fmul_rn(lp[h], sc);
        if (h == hv) sch = sc;
        mr[h] = mn;
        const float p = valid ? ex2(e - mn) : 0.f;
        lp[h] = __fadd_rn(lp[h], p);
        if constexpr (QF) {
          const float pc = pre > 0.f ? p : p * slope;
          lc[h] = __fadd_rn(__fmul_rn(lc[h], sc), pc);
          sP2[wib][h][lane] = make_float2(p, pc);
        } else {
          sPw[wib][h][lane] = p;
        }
      }
      acc = mul4(sch, acc);
      if constexpr (QF) accu = mul4(sch, accu);
      __syncwarp();
      // one gathered row: both accumulations
      auto axpy = [&](int e, const typename SL::raw& r) {
        const float4 x = SL::f(r);
        if constexpr (QF) {
          const float2 pw = sP2[wib][hv][e];
          acc = fma4(pw.x, x, acc);
          accu = fma4(pw.y, x, accu);
        } else {
          acc = fma4(sPw[wib][hv][e], x, acc);
        }
      };
      if (cnt == 32) {
        // full batch: 32/GR groups of GR rows, the next group in flight during this
        // group's FMAs
        constexpr int GR = GRT ? GRT : fwd_group<TP>(), NGR = 32 / GR;
        static_assert(U >= GR, "the prefetch covers the first group");
        const TP* Pl = P + cq;
        typename SL::raw qa[GR], qb[GR];
#pragma unroll
        for (int u = 0; u < GR; ++u) qa[u] = pv[u];  // group 0 was prefetched before the scores
#pragma unroll
        for (int g = 0; g < NGR; g += 2) {
#pragma unroll
          for (int u = 0; u < GR; ++u) {
            const int c = __shfl_sync(FULL, j, GR * g + GR + u);
            qb[u] = SL::load(Pl + ga.row(c) * K, ga.policy(c));
          }
#pragma unroll
          for (int u = 0; u < GR; ++u) axpy(GR * g + u, qa[u]);
          if (g + 2 < NGR) {
#pragma unroll
            for (int u = 0; u < GR; ++u) {
              const int c = __shfl_sync(FULL, j, GR * g + 2 * GR + u);
              qa[u] = SL::load(Pl + ga.row(c) * K, ga.policy(c));
            }
          }
#pragma unroll
          for (int u = 0; u < GR; ++u) axpy(GR * g + GR + u, qb[u]);
        }
      } else {
        for (int k = 0; k < cnt; k += U) {
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int kk = k + u;
            if (k > 0)
              pv[u] = kk < cnt ? SL::load(P + ga.row(sJ[wib][kk]) * K + cq, ga.policy(sJ[wib][kk]))
                               : SL::zero();
          }
#pragma unroll
          for (int u = 0; u < U; ++u)
            if (k + u < cnt) axpy(k + u, pv[u]);
        }
      }
      __syncwarp();
    }
    float l[NH], cs[NH];
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      float x = lp[h], y = lc[h];
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        x += __shfl_xor_sync(FULL, x, off);
        if constexpr (QF) y += __shfl_xor_sync(FULL, y, off);
      }
      l[h] = x;
      cs[h] = y;
    }
    float lh = l[0], ch = cs[0];
#pragma unroll
    for (int h = 1; h < NH; ++h)
      if (h == hv) {
        lh = l[h];
        ch = cs[h];
      }
    if (slot >= 0) {
      st4(o.pacc + slot * K + cq, acc);
      if constexpr (QF) st4(o.pu + slot * K + cq, accu);
      if (lane == 0) {
#pragma unroll
        for (int h = 0; h < NH; ++h) {
          o.pm[slot * NH + h] = mr[h];
          o.pl[slot * NH + h] = l[h];
          if constexpr (QF) o.pc[slot * NH + h] = cs[h];
        }
      }
    } else {
      const float inv = lh > 0.f ? 1.f / lh : 0.f;
      const float4 z = mul4(inv, acc);
      if (o.Z) st4(o.Z + row * K + cq, z);
      st4(o.Hout + row * K + cq, act_fwd4(act, z));
      if constexpr (QF) {
        const float r = lh > 0.f ? ch / lh : 0.f;
        st4(o.Q + row * K + cq, mul4(inv, fma4(-r, acc, accu)));
      }
      if (o.m && lane == 0) {
#pragma unroll
        for (int h = 0; h < NH; ++h) {
          o.m[row * NH + h] = l[h] > 0.f ? mr[h] : 0.f;
          o.l[row * NH + h] = l[h];
        }
      }
    }
  }
}

// BF16 storage (reading B1): the same forward with TWO gathered rows per warp load
// instruction.  A bf16 row of k' = 128 is 256 bytes = 16 lanes x 16 bytes, so the
// half-warps take the even and the odd entries of a batch (lane L: columns
// 8 (L % 16) .. + 7 of entry 2p + L / 16); each half accumulates its entries, and
// the halves are added (one xor-16 shuffle per column) at the end of the item.
// Scores, softmax statistics and outputs are those of gat_fwd_k128_kernel; only
// the summation order of the aggregation differs (even / odd entries, then both).
__device__ __forceinline__ void bf8_to_f8(uint4 u, float (&x)[8]) {
  x[0] = __uint_as_float(u.x << 16);
  x[1] = __uint_as_float(u.x & 0xffff0000u);
  x[2] = __uint_as_float(u.y << 16);
  x[3] = __uint_as_float(u.y & 0xffff0000u);
  x[4] = __uint_as_float(u.z << 16);
  x[5] = __uint_as_float(u.z & 0xffff0000u);
  x[6] = __uint_as_float(u.w << 16);
  x[7] = __uint_as_float(u.w & 0xffff0000u);
}

template <int NH, int UP, int MINB, bool QF>
__global__ void __launch_bounds__(256, MINB)
gat_fwd_k128_pair_kernel(Items it, const bf16* __restrict__ P, const float* __restrict__ st,
                         float slope, int act, GatFwdOut o) {
  constexpr int D = K / NH, LPH = D / 8;  // lanes of a half per head (8 columns each)
  static_assert(D % 8 == 0, "8 columns of one head per lane");
  __shared__ float sPw[QF ? 1 : 8][NH][33];
  __shared__ float2 sP2[QF ? 8 : 1][NH][33];
  __shared__ int sJ[8][32];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int half = lane >> 4, q16 = lane & 15;
  const int hv = q16 / LPH, c8 = q16 * 8;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const Gath ga(it);
  const bf16* Pl = P + c8;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float si[NH], mr[NH], lp[NH], lc[NH];
    load_n<NH>(st + grow * (2 * NH), si);
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      mr[h] = -INFINITY;
      lp[h] = 0.f;
      lc[h] = 0.f;
    }
    float acc[8], accu[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) acc[c] = accu[c] = 0.f;
    int jpre = beg + lane < end ? __ldg(it.col + beg + lane) : 0;
    for (int64_t b0 = beg; b0 < end; b0 += 32) {
      const int cnt = (int)(end - b0 < 32 ? end - b0 : 32);
      const bool valid = lane < cnt;
      const int j = jpre;
      jpre = b0 + 32 + lane < end ? __ldg(it.col + b0 + 32 + lane) : 0;
      sJ[wib][lane] = j;
      __syncwarp();
      auto ld = [&](int e) -> uint4 {
        if (e >= cnt) return make_uint4(0u, 0u, 0u, 0u);
        const int c = sJ[wib][e];
        return ldg16_pol(Pl + ga.row(c) * K, ga.policy(c));
      };
      // the first UP pairs in flight while the scores are computed
      uint4 pv[UP];
#pragma unroll
      for (int u = 0; u < UP; ++u) pv[u] = ld(2 * u + half);
      float tj[NH];
      load_n<NH>(st + ga.row(j) * (2 * NH) + NH, tj, ga.policy(j));
      float sch = 1.f;
#pragma unroll
      for (int h = 0; h < NH; ++h) {
        const float pre = si[h] + tj[h];
        const float e = valid ? fmaxf(pre, slope * pre) : -INFINITY;
        float bm = e;
#pragma unroll
        for (int off = 16; off > 0; off >>= 1) bm = fmaxf(bm, __shfl_xor_sync(FULL, bm, off));
        const float mn = fmaxf(mr[h], bm);
        const float sc = ex2(mr[h] - mn);
        lp[h] = __fmul_rn(lp[h], sc);
        if (h == hv) sch = sc;
        mr[h] = mn;
        const float p = valid ? ex2(e - mn) : 0.f;
        lp[h] = __fadd_rn(lp[h], p);
        if constexpr (QF) {
          const float pc = pre > 0.f ? p : p * slope;
          lc[h] = __fadd_rn(__fmul_rn(lc[h], sc), pc);
          sP2[wib][h][lane] = make_float2(p, pc);
        } else {
          sPw[wib][h][lane] = p;
        }
      }
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        acc[c] *= sch;
        if constexpr (QF) accu[c] *= sch;
      }
      __syncwarp();
      auto axpy = [&](int e, const uint4& r) {
        float x[8];
        bf8_to_f8(r, x);
        if constexpr (QF) {
          const float2 pw = sP2[wib][hv][e];
#pragma unroll
          for (int c = 0; c < 8; ++c) {
            acc[c] = fmaf(pw.x, x[c], acc[c]);
            accu[c] = fmaf(pw.y, x[c], accu[c]);
          }
        } else {
          const float pw = sPw[wib][hv][e];
#pragma unroll
          for (int c = 0; c < 8; ++c) acc[c] = fmaf(pw, x[c], acc[c]);
        }
      };
      if (cnt == 32) {
        // 16 pairs: groups of UP pairs, the next group in flight during this one
        constexpr int NG = 16 / UP;
        uint4 qa[UP], qb[UP];
#pragma unroll
        for (int u = 0; u < UP; ++u) qa[u] = pv[u];
#pragma unroll
        for (int g = 0; g < NG; g += 2) {
#pragma unroll
          for (int u = 0; u < UP; ++u) qb[u] = ld(2 * (UP * (g + 1) + u) + half);
#pragma unroll
          for (int u = 0; u < UP; ++u) axpy(2 * (UP * g + u) + half, qa[u]);
          if (g + 2 < NG) {
#pragma unroll
            for (int u = 0; u < UP; ++u) qa[u] = ld(2 * (UP * (g + 2) + u) + half);
          }
#pragma unroll
          for (int u = 0; u < UP; ++u) axpy(2 * (UP * (g + 1) + u) + half, qb[u]);
        }
      } else {
        const int npair = (cnt + 1) >> 1;
        for (int k0 = 0; k0 < npair; k0 += UP) {
          if (k0 > 0) {
#pragma unroll
            for (int u = 0; u < UP; ++u) pv[u] = ld(2 * (k0 + u) + half);
          }
#pragma unroll
          for (int u = 0; u < UP; ++u) {
            const int e = 2 * (k0 + u) + half;
            if (e < cnt) axpy(e, pv[u]);
          }
        }
      }
      __syncwarp();
    }
    // the two halves' partial sums (even / odd entries)
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      acc[c] += __shfl_xor_sync(FULL, acc[c], 16);
      if constexpr (QF) accu[c] += __shfl_xor_sync(FULL, accu[c], 16);
    }
    float l[NH], cs[NH];
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      float x = lp[h], y = lc[h];
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) {
        x += __shfl_xor_sync(FULL, x, off);
        if constexpr (QF) y += __shfl_xor_sync(FULL, y, off);
      }
      l[h] = x;
      cs[h] = y;
    }
    float lh = l[0], ch = cs[0];
#pragma unroll
    for (int h = 1; h < NH; ++h)
      if (h == hv) {
        lh = l[h];
        ch = cs[h];
      }
    // lane L stores columns c8 + 4 (L / 16) .. + 3
    const int co = c8 + 4 * half;
    const float4 a4 = half ? make_float4(acc[4], acc[5], acc[6], acc[7])
                           : make_float4(acc[0], acc[1], acc[2], acc[3]);
    const float4 u4 = half ? make_float4(accu[4], accu[5], accu[6], accu[7])
                           : make_float4(accu[0], accu[1], accu[2], accu[3]);
    if (slot >= 0) {
      st4(o.pacc + slot * K + co, a4);
      if constexpr (QF) st4(o.pu + slot * K + co, u4);
      if (lane == 0) {
#pragma unroll
        for (int h = 0; h < NH; ++h) {
          o.pm[slot * NH + h] = mr[h];
          o.pl[slot * NH + h] = l[h];
          if constexpr (QF) o.pc[slot * NH + h] = cs[h];
        }
      }
    } else {
      const float inv = lh > 0.f ? 1.f / lh : 0.f;
      const float4 z = mul4(inv, a4);
      if (o.Z) st4(o.Z + row * K + co, z);
      st4(o.Hout + row * K + co, act_fwd4(act, z));
      if constexpr (QF) {
        const float r = lh > 0.f ? ch / lh : 0.f;
        st4(o.Q + row * K + co, mul4(inv, fma4(-r, a4, u4)));
      }
      if (o.m && lane == 0) {
#pragma unroll
        for (int h = 0; h < NH; ++h) {
          o.m[row * NH + h] = l[h] > 0.f ? mr[h] : 0.f;
          o.l[row * NH + h] = l[h];
        }
      }
    }
  }
}

// ---------------------------------------------------------------- backward
template <typename TP, int B>
struct BwdBatch {  // operands of one batch of B edges held by one lane (raw slices)
  typename Slice<TP>::raw Pi[B], Gi[B];
  float4 ri;
  float ti;
};

template <typename TP, int NH, int B, int MINB>
__global__ void __launch_bounds__(256, MINB)
gat_bwd_k128_kernel(Items it, GatBwdArgs A) {
  constexpr int D = K / NH, HL = D / 4;
  static_assert(B <= HL && (B & (B - 1)) == 0, "B edges per batch, at most one per head lane");
  using TR = Transpose<B>;
  const int lane = threadIdx.x & 31;
  const int hv = lane / HL, ql = lane % HL, cq = lane * 4, gbase = lane & ~(HL - 1);
  const int my_b = TR::edge_of(ql);
  const bool owner = (ql >> TR::T) == 0;  // lanes beyond the first B of a group hold duplicates
  const float slope = A.slope;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const TP* Pb = pick<TP>(A.P, A.P16);
  const TP* Gb = pick<TP>(A.G, A.G16);
  const TP* Pl = Pb + cq;
  const TP* Gl = Gb + cq;
  float4 da1 = f4(0.f), da2 = f4(0.f);
  const Gath ga(it);

  for (int64_t w = gw; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    const float4 Pj = ldg4(Pb + grow * K + cq);
    const float4 Gj = ldg4(Gb + grow * K + cq);
    const float4 rj = __ldg(A.rec + grow * NH + hv);        // {s_j, m_j, 1/l_j, delta_j}
    const float tj = __ldg(A.st + grow * (2 * NH) + NH + hv);
    float4 acc = f4(0.f);
    float dsp = 0.f, dtp = 0.f;
    // gathers of batch (window offset off, cnt valid edges): rows i of P, G and the
    // record of the edge this lane owns after the reduction
    using SL = Slice<TP>;
    auto load = [&](BwdBatch<TP, B>& q, int cidx, int off, int cnt) {
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const int c = __shfl_sync(FULL, cidx, off + b);
        if (b < cnt) {
          const int64_t i = ga.row(c);
          const uint64_t pol = ga.policy(c);
          q.Pi[b] = SL::load(Pl + i * K, pol);
          q.Gi[b] = SL::load(Gl + i * K, pol);
        } else {
          q.Pi[b] = q.Gi[b] = SL::zero();
        }
      }
      const int cm = __shfl_sync(FULL, cidx, off + my_b);
      const bool vm = my_b < cnt;
      const int64_t im = ga.row(cm);
      const uint64_t polm = ga.policy(cm);
      q.ri = vm ? ldg4_pol(reinterpret_cast<const float*>(A.rec + im * NH + hv), polm) : f4(0.f);
      q.ti = vm ? ldg1_pol(A.st + im * (2 * NH) + NH + hv, polm) : 0.f;
    };
    auto body = [&](const BwdBatch<TP, B>& q, int cnt) {
      float x1[B], x2[B];
#pragma unroll
      for (int b = 0; b < B; ++b) {
        x1[b] = dot4(Gj, SL::f(q.Pi[b]));  // G_j . P_i  (row role)
        x2[b] = dot4(SL::f(q.Gi[b]), Pj);  // G_i . P_j  (column role)
      }
      TR::template reduce<HL>(x1, lane);
      TR::template reduce<HL>(x2, lane);
      const bool vm = my_b < cnt;
      // row role: entry (j,i) of row j
      const float pre = rj.x + q.ti;
      const float e = fmaxf(pre, slope * pre);
      const float aji = ex2(e - rj.y) * rj.z;
      const float dcji = aji * (pre > 0.f ? 1.f : slope) * (x1[0] - rj.w);
      // column role: entry (i,j) of row i
      const float pre2 = q.ri.x + tj;
      const float e2 = fmaxf(pre2, slope * pre2);
      float aij = ex2(e2 - q.ri.y) * q.ri.z;
      const float dcij = aij * (pre2 > 0.f ? 1.f : slope) * (x2[0] - q.ri.w);
      if (vm && owner) {
        dsp += dcji;
        dtp += dcij;
      }
      if (!vm) aij = 0.f;
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const float ab = __shfl_sync(FULL, aij, gbase + TR::lane_of(b));
        acc = fma4(ab, SL::f(q.Gi[b]), acc);
      }
    };
    // column ids one window ahead: the next window's ids load during this window
    int cpre = beg + lane < end ? __ldg(it.col + beg + lane) : 0;
    for (int64_t w0 = beg; w0 < end; w0 += 32) {
      const int wcnt = (int)(end - w0 < 32 ? end - w0 : 32);
      const int cidx = cpre;
      cpre = w0 + 32 + lane < end ? __ldg(it.col + w0 + 32 + lane) : 0;
      if (wcnt == 32) {
        // full window: 32/B batches, the next batch's gathers in flight during this one
        BwdBatch<TP, B> qa, qb;
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
          BwdBatch<TP, B> q;
          const int cnt = wcnt - off < B ? wcnt - off : B;
          load(q, cidx, off, cnt);
          body(q, cnt);
        }
      }
    }
    // per-head row sums ds_j, dt_j: every lane of the head group ends with the total
#pragma unroll
    for (int o = 1; o < HL; o <<= 1) {
      dsp += __shfl_xor_sync(FULL, dsp, o);
      dtp += __shfl_xor_sync(FULL, dtp, o);
    }
    if (slot >= 0) {
      st4(A.pacc + slot * K + cq, acc);
      if (ql == 0) {
        A.pds[slot * NH + hv] = dsp;
        A.pdt[slot * NH + hv] = dtp;
      }
    } else {
      const float4 a1v = ldg4(A.a + hv * 2 * D + cq % D);
      const float4 a2v = ldg4(A.a + hv * 2 * D + D + cq % D);
      float4 dp = fma4(dsp, a1v, acc);
      dp = fma4(dtp, a2v, dp);
      st4(A.dP + row * K + cq, dp);
      da1 = fma4(dsp, Pj, da1);
      da2 = fma4(dtp, Pj, da2);
    }
  }
  st4(A.da_part + gw * 2 * K + cq, da1);
  st4(A.da_part + gw * 2 * K + K + cq, da2);
}

// ---------------------------------------------------------------- factored backward
// Column role only (the row role's ds_j = G_j . Q_j comes from the prologue,
// gat_args.cuh): per row j, edges in windows of 32 (one edge per lane) —
//   lane e: rec_i of all heads -> alpha_ij = 2^(LReLU(s_i + t_j) - m_i) / l_i,
//   c'_ij = alpha_ij lambda_ij, partial sums of c'_ij delta_i;
//   then the warp walks the window: lane q owns columns 4q..4q+3 of G_i and
//   accumulates acc_j += alpha_ij G_i and v_j += c'_ij G_i (16-byte gather, 8 FMAs).
// Per row: dt_j = P_j . v_j - sum_i c'_ij delta_i, dP_j = acc_j + ds_j a1 + dt_j a2.
// Per edge it moves the index, one G row and the NH records (4 + K f + 16 NH bytes).
template <typename TP, int NH, int MINB, int GRT = 0>
__global__ void __launch_bounds__(256, MINB)
gat_bwd_k128f_kernel(Items it, GatBwdArgs A) {
  constexpr int D = K / NH, HL = D / 4;
  __shared__ float2 sAC[8][NH][33];  // {alpha_ij, c'_ij}
  __shared__ int sJ[8][32];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int hv = lane / HL, cq = lane * 4;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const TP* Pb = pick<TP>(A.P, A.P16);
  const TP* Gb = pick<TP>(A.G, A.G16);
  const float slope = A.slope;
  const Gath ga(it);
  using SL = Slice<TP>;
  float4 da1 = f4(0.f), da2 = f4(0.f);
  for (int64_t w = gw; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float tj[NH], sd[NH];
    load_n<NH>(A.st + grow * (2 * NH) + NH, tj);
#pragma unroll
    for (int h = 0; h < NH; ++h) sd[h] = 0.f;
    float4 acc = f4(0.f), accv = f4(0.f);
    int jpre = beg + lane < end ? __ldg(it.col + beg + lane) : 0;
    for (int64_t b0 = beg; b0 < end; b0 += 32) {
      const int cnt = (int)(end - b0 < 32 ? end - b0 : 32);
      const bool valid = lane < cnt;
      const int j = jpre;
      jpre = b0 + 32 + lane < end ? __ldg(it.col + b0 + 32 + lane) : 0;
      sJ[wib][lane] = j;
      __syncwarp();
      constexpr int GR = GRT ? GRT : fwd_group<TP>(), NGR = 32 / GR;
      typename SL::raw qa[GR], qb[GR];
      // the first group of G rows is in flight while the weights are computed
#pragma unroll
      for (int u = 0; u < GR; ++u)
        qa[u] = u < cnt ? SL::load(Gb + ga.row(sJ[wib][u]) * K + cq, ga.policy(sJ[wib][u]))
                        : SL::zero();
      {
        const int64_t ir = ga.row(j);
        const uint64_t pol = ga.policy(j);
#pragma unroll
        for (int h = 0; h < NH; ++h) {
          const float4 r = valid ? ldg4_pol(reinterpret_cast<const float*>(A.rec + ir * NH + h), pol)
                                 : f4(0.f);  // {s_i, m_i, 1/l_i, delta_i}
          const float pre = r.x + tj[h];
          const float e = fmaxf(pre, slope * pre);
          const float al = valid ? ex2(e - r.y) * r.z : 0.f;
          const float cc = pre > 0.f ? al : al * slope;
          sd[h] = fmaf(cc, r.w, sd[h]);
          sAC[wib][h][lane] = make_float2(al, cc);
        }
      }
      __syncwarp();
      auto axpy = [&](int e, const typename SL::raw& r) {
        const float4 x = SL::f(r);
        const float2 ac = sAC[wib][hv][e];
        acc = fma4(ac.x, x, acc);
        accv = fma4(ac.y, x, accv);
      };
      const TP* Gl = Gb + cq;
      if (cnt == 32) {
#pragma unroll
        for (int g = 0; g < NGR; g += 2) {
#pragma unroll
          for (int u = 0; u < GR; ++u) {
            const int c = __shfl_sync(FULL, j, GR * g + GR + u);
            qb[u] = SL::load(Gl + ga.row(c) * K, ga.policy(c));
          }
#pragma unroll
          for (int u = 0; u < GR; ++u) axpy(GR * g + u, qa[u]);
          if (g + 2 < NGR) {
#pragma unroll
            for (int u = 0; u < GR; ++u) {
              const int c = __shfl_sync(FULL, j, GR * g + 2 * GR + u);
              qa[u] = SL::load(Gl + ga.row(c) * K, ga.policy(c));
            }
          }
#pragma unroll
          for (int u = 0; u < GR; ++u) axpy(GR * g + GR + u, qb[u]);
        }
      } else {
        for (int k = 0; k < cnt; k += GR) {
          if (k > 0) {
#pragma unroll
            for (int u = 0; u < GR; ++u) {
              const int kk = k + u;
              qa[u] = kk < cnt ? SL::load(Gl + ga.row(sJ[wib][kk]) * K, ga.policy(sJ[wib][kk]))
                               : SL::zero();
            }
          }
#pragma unroll
          for (int u = 0; u < GR; ++u)
            if (k + u < cnt) axpy(k + u, qa[u]);
        }
      }
      __syncwarp();
    }
    // per row: dt_j = P_j . v_j - sum_i c'_ij delta_i  (head of lane hv)
    const float4 Pj = SL::f(SL::load(Pb + grow * K + cq));
    float x = dot4(Pj, accv);
#pragma unroll
    for (int o = 1; o < HL; o <<= 1) x += __shfl_xor_sync(FULL, x, o);
    float sdh = 0.f;
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      float y = sd[h];
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) y += __shfl_xor_sync(FULL, y, off);
      if (h == hv) sdh = y;
    }
    const float dt = x - sdh;
    if (slot >= 0) {
      st4(A.pacc + slot * K + cq, acc);
      if ((lane % HL) == 0) {
        A.pdt[slot * NH + hv] = dt;
        A.pds[slot * NH + hv] = it.chunk_idx[slot] == 0 ? A.ds_row[row * NH + hv] : 0.f;
      }
    } else {
      const float ds = A.ds_row[row * NH + hv];
      const float4 a1v = ldg4(A.a + hv * 2 * D + cq % D);
      const float4 a2v = ldg4(A.a + hv * 2 * D + D + cq % D);
      float4 dp = fma4(ds, a1v, acc);
      dp = fma4(dt, a2v, dp);
      st4(A.dP + row * K + cq, dp);
      da1 = fma4(ds, Pj, da1);
      da2 = fma4(dt, Pj, da2);
    }
  }
  st4(A.da_part + gw * 2 * K + cq, da1);
  st4(A.da_part + gw * 2 * K + K + cq, da2);
}

// BF16 storage: the factored backward with two gathered G rows per warp load
// instruction (the pairing of gat_fwd_k128_pair_kernel: half-warps take the even /
// odd entries, 8 columns per lane, halves added at the end of the item).  Lane L
// owns output columns co = 8 (L % 16) + 4 (L / 16) .. + 3 for dP, the chunk partials
// and its da partial.
template <int NH, int UP, int MINB>
__global__ void __launch_bounds__(256, MINB)
gat_bwd_k128f_pair_kernel(Items it, GatBwdArgs A) {
  constexpr int D = K / NH, LPH = D / 8;
  static_assert(D % 8 == 0, "8 columns of one head per lane");
  __shared__ float2 sAC[8][NH][33];  // {alpha_ij, c'_ij}
  __shared__ int sJ[8][32];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int half = lane >> 4, q16 = lane & 15;
  const int hv = q16 / LPH, c8 = q16 * 8, co = c8 + 4 * half;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const bf16* Gl = A.G16 + c8;
  const float slope = A.slope;
  const Gath ga(it);
  using SL = Slice<bf16>;
  float4 da1 = f4(0.f), da2 = f4(0.f);
  for (int64_t w = gw; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float tj[NH], sd[NH];
    load_n<NH>(A.st + grow * (2 * NH) + NH, tj);
#pragma unroll
    for (int h = 0; h < NH; ++h) sd[h] = 0.f;
    float acc[8], accv[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) acc[c] = accv[c] = 0.f;
    int jpre = beg + lane < end ? __ldg(it.col + beg + lane) : 0;
    for (int64_t b0 = beg; b0 < end; b0 += 32) {
      const int cnt = (int)(end - b0 < 32 ? end - b0 : 32);
      const bool valid = lane < cnt;
      const int j = jpre;
      jpre = b0 + 32 + lane < end ? __ldg(it.col + b0 + 32 + lane) : 0;
      sJ[wib][lane] = j;
      __syncwarp();
      auto ld = [&](int e) -> uint4 {
        if (e >= cnt) return make_uint4(0u, 0u, 0u, 0u);
        const int c = sJ[wib][e];
        return ldg16_pol(Gl + ga.row(c) * K, ga.policy(c));
      };
      uint4 qa[UP], qb[UP];
      // the first group of G row pairs is in flight while the weights are computed
#pragma unroll
      for (int u = 0; u < UP; ++u) qa[u] = ld(2 * u + half);
      {
        const int64_t ir = ga.row(j);
        const uint64_t pol = ga.policy(j);
#pragma unroll
        for (int h = 0; h < NH; ++h) {
          const float4 r = valid ? ldg4_pol(reinterpret_cast<const float*>(A.rec + ir * NH + h), pol)
                                 : f4(0.f);  // {s_i, m_i, 1/l_i, delta_i}
          const float pre = r.x + tj[h];
          const float e = fmaxf(pre, slope * pre);
          const float al = valid ? ex2(e - r.y) * r.z : 0.f;
          const float cc = pre > 0.f ? al : al * slope;
          sd[h] = fmaf(cc, r.w, sd[h]);
          sAC[wib][h][lane] = make_float2(al, cc);
        }
      }
      __syncwarp();
      auto axpy = [&](int e, const uint4& r) {
        float x[8];
        bf8_to_f8(r, x);
        const float2 ac = sAC[wib][hv][e];
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          acc[c] = fmaf(ac.x, x[c], acc[c]);
          accv[c] = fmaf(ac.y, x[c], accv[c]);
        }
      };
      if (cnt == 32) {
        constexpr int NG = 16 / UP;
#pragma unroll
        for (int g = 0; g < NG; g += 2) {
#pragma unroll
          for (int u = 0; u < UP; ++u) qb[u] = ld(2 * (UP * (g + 1) + u) + half);
#pragma unroll
          for (int u = 0; u < UP; ++u) axpy(2 * (UP * g + u) + half, qa[u]);
          if (g + 2 < NG) {
#pragma unroll
            for (int u = 0; u < UP; ++u) qa[u] = ld(2 * (UP * (g + 2) + u) + half);
          }
#pragma unroll
          for (int u = 0; u < UP; ++u) axpy(2 * (UP * (g + 1) + u) + half, qb[u]);
        }
      } else {
        const int npair = (cnt + 1) >> 1;
        for (int k0 = 0; k0 < npair; k0 += UP) {
          if (k0 > 0) {
#pragma unroll
            for (int u = 0; u < UP; ++u) qa[u] = ld(2 * (k0 + u) + half);
          }
#pragma unroll
          for (int u = 0; u < UP; ++u) {
            const int e = 2 * (k0 + u) + half;
            if (e < cnt) axpy(e, qa[u]);
          }
        }
      }
      __syncwarp();
    }
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      acc[c] += __shfl_xor_sync(FULL, acc[c], 16);
      accv[c] += __shfl_xor_sync(FULL, accv[c], 16);
    }
    const float4 a4 = half ? make_float4(acc[4], acc[5], acc[6], acc[7])
                           : make_float4(acc[0], acc[1], acc[2], acc[3]);
    const float4 v4 = half ? make_float4(accv[4], accv[5], accv[6], accv[7])
                           : make_float4(accv[0], accv[1], accv[2], accv[3]);
    // per row: dt_j = P_j . v_j - sum_i c'_ij delta_i (head hv: lanes 4hv.. of both halves)
    const float4 Pj = SL::f(SL::load(A.P16 + grow * K + co));
    float x = dot4(Pj, v4);
#pragma unroll
    for (int o = 1; o < LPH; o <<= 1) x += __shfl_xor_sync(FULL, x, o);
    x += __shfl_xor_sync(FULL, x, 16);
    float sdh = 0.f;
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      float y = sd[h];
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) y += __shfl_xor_sync(FULL, y, off);
      if (h == hv) sdh = y;
    }
    const float dt = x - sdh;
    if (slot >= 0) {
      st4(A.pacc + slot * K + co, a4);
      if (half == 0 && (q16 % LPH) == 0) {
        A.pdt[slot * NH + hv] = dt;
        A.pds[slot * NH + hv] = it.chunk_idx[slot] == 0 ? A.ds_row[row * NH + hv] : 0.f;
      }
    } else {
      const float ds = A.ds_row[row * NH + hv];
      const float4 a1v = ldg4(A.a + hv * 2 * D + co % D);
      const float4 a2v = ldg4(A.a + hv * 2 * D + D + co % D);
      float4 dp = fma4(ds, a1v, a4);
      dp = fma4(dt, a2v, dp);
      st4(A.dP + row * K + co, dp);
      da1 = fma4(ds, Pj, da1);
      da2 = fma4(dt, Pj, da2);
    }
  }
  st4(A.da_part + gw * 2 * K + co, da1);
  st4(A.da_part + gw * 2 * K + K + co, da2);
}

template <typename F>
int grid_for(F* f) {
  return persistent_blocks(reinterpret_cast<const void*>(f));
}

}  // namespace

bool gat_k128_supported(int k_out, int heads) {
  return k_out == 128 && (heads == 1 || heads == 2 || heads == 4 || heads == 8);
}

#define AGNN_K128_DISPATCH(NH_, CALL)                                   \
  do {                                                                  \
    if (NH_ == 1) { constexpr int NH = 1; CALL; }                       \
    else if (NH_ == 2) { constexpr int NH = 2; CALL; }                  \
    else if (NH_ == 4) { constexpr int NH = 4; CALL; }                  \
    else if (NH_ == 8) { constexpr int NH = 8; CALL; }                  \
    else return fail(AGNN_EUNSUPPORTED, "GAT k'=128: heads must be 1/2/4/8"); \
  } while (0)

template <int NH>
constexpr int bwd_batch() { return (K / NH / 4) >= 4 ? 4 : K / NH / 4; }
// bf16 rows are half the bytes: 8 edges per batch (one per lane of a head group
// when HL = 8) keep as many bytes in flight per lane as 4 fp32 edges
template <int NH>
constexpr int bwd_batch_bf16() { return (K / NH / 4) >= 8 ? 8 : K / NH / 4; }

agnn_status gat_fwd_k128(const Items& it_all, int heads, const float* P, const float* st,
                         float slope, int act, const GatFwdOut& o, cudaStream_t s) {
  agnn_status sst = (gat_bundles_enabled(it_all, false) && it_all.bundles)
                        ? gat_fwd_bundle<float>(it_all, heads, P, st, slope, act, o, s)
                        : gat_fwd_short<float>(it_all, heads, P, st, slope, act, o, s);
  if (sst != AGNN_OK) return sst;
  const Items it = long_items(it_all);
  if (it.n_chunks + it.n_light == 0) return AGNN_OK;
  AGNN_K128_DISPATCH(heads, ({
    // 3 blocks / SM, 4-row gather groups (measured C5, round 1: 2 blocks / SM with
    // 8-row groups and 4 blocks / SM were both slower)
    auto* kern = o.Q ? gat_fwd_k128_kernel<float, NH, 4, 3, true>
                     : gat_fwd_k128_kernel<float, NH, 4, 3, false>;
    kern<<<grid_for(kern), 256, 0, s>>>(it, P, st, slope, act, o);
    AGNN_LAUNCH_CHECK("gat_fwd_kernel");
  }));
  return AGNN_OK;
}

agnn_status gat_fwd_k128_bf16(const Items& it_all, int heads, const bf16* P, const float* st,
                              float slope, int act, const GatFwdOut& o, cudaStream_t s) {
  agnn_status sst = (gat_bundles_enabled(it_all, true) && it_all.bundles)
                        ? gat_fwd_bundle<bf16>(it_all, heads, P, st, slope, act, o, s)
                        : gat_fwd_short<bf16>(it_all, heads, P, st, slope, act, o, s);
  if (sst != AGNN_OK) return sst;
  const Items it = long_items(it_all);
  if (it.n_chunks + it.n_light == 0) return AGNN_OK;
  AGNN_K128_DISPATCH(heads, ({
    // two rows per load instruction, 3 blocks / SM (measured C5 bf16: 53.3 -> 47.2 ms
    // against gat_fwd_k128_kernel<bf16> with 8-row groups)
    auto* kern = o.Q ? gat_fwd_k128_pair_kernel<NH, 4, 3, true>
                     : gat_fwd_k128_pair_kernel<NH, 4, 3, false>;
    kern<<<grid_for(kern), 256, 0, s>>>(it, P, st, slope, act, o);
    AGNN_LAUNCH_CHECK("gat_fwd_kernel");
  }));
  return AGNN_OK;
}

agnn_status gat_bwd_k128(const Items& it_all, int heads, const GatBwdArgs& A, int64_t* warps,
                         cudaStream_t s) {
  *warps = 0;
  const Items it = long_items(it_all);
  AGNN_K128_DISPATCH(heads, ({
    constexpr int B = bwd_batch<NH>();
    constexpr int B16 = bwd_batch_bf16<NH>();
    int grid;
    if (A.P16) {  // BF16 mode (reading B1)
      grid = grid_for(gat_bwd_k128_kernel<bf16, NH, B16, 2>);
      gat_bwd_k128_kernel<bf16, NH, B16, 2><<<grid, 256, 0, s>>>(it, A);
    } else {
      grid = grid_for(gat_bwd_k128_kernel<float, NH, B, 2>);
      gat_bwd_k128_kernel<float, NH, B, 2><<<grid, 256, 0, s>>>(it, A);
    }
    AGNN_LAUNCH_CHECK("gat_bwd_kernel");
    *warps = (int64_t)grid * 8;
  }));
  // short rows: their da partials follow the main kernel's rows
  int64_t sw = 0;
  agnn_status sst = gat_bwd_short(it_all, heads, A, *warps, &sw, s);
  *warps += sw;
  return sst;
}

agnn_status gat_bwd_k128f(const Items& it_all, int heads, const GatBwdArgs& A, int64_t* warps,
                          cudaStream_t s) {
  *warps = 0;
  const Items it = long_items(it_all);
  AGNN_K128_DISPATCH(heads, ({
    // fp32: 2 blocks / SM (measured C5, round 1: 73.5 -> 69.2 ms against 3 blocks);
    // bf16: two G rows per load instruction, 2 blocks / SM (C5: 58.6 -> 51.8 ms against
    // gat_bwd_k128f_kernel<bf16> at 3 blocks; the pair kernel at 3 blocks spills, 55.3)
    auto* kern = A.P16 ? (void (*)(Items, GatBwdArgs))gat_bwd_k128f_pair_kernel<NH, 4, 2>
                       : (void (*)(Items, GatBwdArgs))gat_bwd_k128f_kernel<float, NH, 2>;
    const int grid = grid_for(kern);
    kern<<<grid, 256, 0, s>>>(it, A);
    AGNN_LAUNCH_CHECK("gat_bwd_kernel");
    *warps = (int64_t)grid * 8;
  }));
  // short rows: their da partials follow the main kernel's rows
  int64_t sw = 0;
  agnn_status sst = (gat_bundles_enabled(it_all, A.P16 != nullptr) && it_all.bundles)
                        ? gat_bwd_bundle(it_all, heads, A, *warps, &sw, s)
                        : gat_bwd_short_f(it_all, heads, A, *warps, &sw, s);
  *warps += sw;
  return sst;
}

}  // namespace agnn
