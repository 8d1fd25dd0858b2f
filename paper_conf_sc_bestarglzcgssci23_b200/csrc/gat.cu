// gat.cu — fused sparse kernels of the GAT layer (forward and backward).
//
// Forward (PAPER.md:177 Psi = sm(A (.) LReLU(C)), C = s 1^T + 1 t^T, and the
// SpMM Z = Psi P with P = H W), one pass over the CSR:
//   per row i and head h: online (flash-style) softmax over the stored entries
//   e_ij = LReLU(s_i + t_j), Z_i = sum_j alpha_ij P_j, H_out = sigma(Z)  —  the
//   n x n virtual C and the sparse Psi are never stored.
// Backward (Eq. 6 with Psi^T, readings A11/A12): one pass
// over the symmetric CSR handles both roles of every stored entry (j,i):
//   row role    dc_ji = alpha_ji (G_j.P_i - delta_j) lambda_ji   -> ds_j
//   column role dc_ij = alpha_ij (G_i.P_j - delta_i) lambda_ij   -> dt_j,
//               acc_j += alpha_ij G_i
//   dP_j = acc_j + ds_j a1 + dt_j a2 ;  da1 += ds_j P_j ; da2 += dt_j P_j
// with alpha recomputed from the saved row statistics (m, 1/l) — no attention
// matrix is ever stored.
//
// Work decomposition: persistent warps walk a static item list (heavy-row
// chunks first, then light rows); a warp owns one row (or one <= chunk-edge
// slice of a heavy row) at a time; lanes own 128-bit column slices of the
// feature rows; sub-warp lane groups split the edges when K < 128.  Heavy-row
// chunks write (m, l, acc) partials merged in ascending chunk order, so the
// result does not depend on launch geometry or on the number of GPUs.
#include <cfloat>

#include "gat_args.cuh"

namespace agnn {

namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr float NEG_INF = -INFINITY;

using FwdOut = GatFwdOut;

__device__ __forceinline__ void merge_softmax(float& m, float& l, float4& acc, float m2, float l2,
                                              float4 acc2) {
  const float mn = fmaxf(m, m2);
  if (mn == NEG_INF) return;
  const float x = ex2(m - mn), y = ex2(m2 - mn);
  l = fmaf(l, x, l2 * y);  // explicit: no contraction choice left to the compiler
  acc = make_float4(fmaf(acc.x, x, acc2.x * y), fmaf(acc.y, x, acc2.y * y),
                    fmaf(acc.z, x, acc2.z * y), fmaf(acc.w, x, acc2.w * y));
  m = mn;
}

template <int K, int NH>
__device__ __forceinline__ void item_range(const Items& it, int64_t w, int64_t& row, int64_t& beg,
                                           int64_t& end, int64_t& slot) {
  if (w < it.n_chunks) {
    row = it.chunk_row[w];
    beg = it.row_ptr[row] + (int64_t)it.chunk_idx[w] * it.chunk;
    end = min(beg + (int64_t)it.chunk, it.row_ptr[row + 1]);
    slot = w;
  } else {
    row = it.light_rows[w - it.n_chunks];
    beg = it.row_ptr[row];
    end = it.row_ptr[row + 1];
    slot = -1;
  }
}

template <int K, int NH>
__device__ __forceinline__ void fwd_finish(int64_t row, const float (&m)[RowLayout<K, NH>::VPL],
                                           const float (&l)[RowLayout<K, NH>::VPL],
                                           const float4 (&acc)[RowLayout<K, NH>::VPL], int q, int act,
                                           const FwdOut& o) {
  using L = RowLayout<K, NH>;
#pragma unroll
  for (int v = 0; v < L::VPL; ++v) {
    const int c = L::col(v, q);
    const float inv = l[v] > 0.f ? 1.f / l[v] : 0.f;
    const float4 z = mul4(inv, acc[v]);
    if (o.Z) st4(o.Z + row * K + c, z);
    st4(o.Hout + row * K + c, act_fwd4(act, z));
    if (o.m && (c % L::D) == 0) {
      o.m[row * NH + c / L::D] = (l[v] > 0.f) ? m[v] : 0.f;
      o.l[row * NH + c / L::D] = l[v];
    }
  }
}

// ---------------------------------------------------------------- forward
// merge of two online-softmax states that also carry the factored backward's
// (lc, accu) = (sum p lambda, sum p lambda P) with the same rescale factors
__device__ __forceinline__ void merge_softmax_q(float& m, float& l, float4& acc, float& lc,
                                                float4& accu, float m2, float l2, float4 acc2,
                                                float lc2, float4 accu2) {
  const float mn = fmaxf(m, m2);
  if (mn == NEG_INF) return;
  const float x = ex2(m - mn), y = ex2(m2 - mn);
  l = fmaf(l, x, l2 * y);
  acc = make_float4(fmaf(acc.x, x, acc2.x * y), fmaf(acc.y, x, acc2.y * y),
                    fmaf(acc.z, x, acc2.z * y), fmaf(acc.w, x, acc2.w * y));
  lc = fmaf(lc, x, lc2 * y);
  accu = make_float4(fmaf(accu.x, x, accu2.x * y), fmaf(accu.y, x, accu2.y * y),
                     fmaf(accu.z, x, accu2.z * y), fmaf(accu.w, x, accu2.w * y));
  m = mn;
}

// QF (training, factored backward; gat_args.cuh): also u_i = sum_j c_ij P_j and
// C_i = sum_j c_ij (c = p lambda) with the same rescaling; Q_i = (u - (C/l) acc) / l.
template <int K, int NH, int U, bool QF>
__global__ void __launch_bounds__(kSparseThreads)
gat_fwd_kernel(Items it, const float* __restrict__ P, const float* __restrict__ st, float slope,
               int act, FwdOut o) {
  using L = RowLayout<K, NH>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_range<K, NH>(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float si[L::VPL], m[L::VPL], l[L::VPL], lc[L::VPL];
    float4 acc[L::VPL], accu[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      si[v] = __ldg(st + grow * (2 * NH) + L::head(v, q));
      m[v] = NEG_INF;
      l[v] = lc[v] = 0.f;
      acc[v] = accu[v] = f4(0.f);
    }
    for (int64_t e0 = beg; e0 < end; e0 += 32) {
      const int cnt = (int)(end - e0 < 32 ? end - e0 : 32);
      const int myc = lane < cnt ? __ldg(it.col + e0 + lane) : 0;
      for (int b = 0; b < cnt; b += L::GROUPS * U) {
        float4 pj[U][L::VPL];
        float tj[U][L::VPL];
        bool val[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int se = b + u * L::GROUPS + g;
          val[u] = se < cnt;
          const int64_t j = __shfl_sync(FULL, myc, se & 31);
#pragma unroll
          for (int v = 0; v < L::VPL; ++v) {
            if (val[u]) {
              pj[u][v] = ldg4(P + j * K + L::col(v, q));
              tj[u][v] = __ldg(st + j * (2 * NH) + NH + L::head(v, q));
            } else {
              pj[u][v] = f4(0.f);
              tj[u][v] = 0.f;
            }
          }
        }
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) {
          float ev[U], pre[U];
          float mn = m[v];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            pre[u] = si[v] + tj[u][v];
            ev[u] = pre[u] > 0.f ? pre[u] : slope * pre[u];
            if (val[u]) mn = fmaxf(mn, ev[u]);
          }
          if (mn != NEG_INF) {
            const float sc = ex2(m[v] - mn);
            // rounded mul / add, never contracted: the QF and inference variants agree
            // bitwise, and lc follows the same operations as l
            l[v] = __fmul_rn(l[v], sc);
            acc[v] = mul4(sc, acc[v]);
            if constexpr (QF) {
              lc[v] = __fmul_rn(lc[v], sc);
              accu[v] = mul4(sc, accu[v]);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
              if (val[u]) {
                const float p = ex2(ev[u] - mn);
                l[v] = __fadd_rn(l[v], p);
                acc[v] = fma4(p, pj[u][v], acc[v]);
                if constexpr (QF) {
                  const float pc = pre[u] > 0.f ? p : p * slope;
                  lc[v] = __fadd_rn(lc[v], pc);
                  accu[v] = fma4(pc, pj[u][v], accu[v]);
                }
              }
            }
            m[v] = mn;
          }
        }
      }
    }
    // merge the lane groups (ascending butterfly)
#pragma unroll
    for (int off = L::LANES; off < 32; off <<= 1) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        const float m2 = __shfl_xor_sync(FULL, m[v], off), l2 = __shfl_xor_sync(FULL, l[v], off);
        float4 a2, u2 = f4(0.f);
        float lc2 = 0.f;
        a2.x = __shfl_xor_sync(FULL, acc[v].x, off);
        a2.y = __shfl_xor_sync(FULL, acc[v].y, off);
        a2.z = __shfl_xor_sync(FULL, acc[v].z, off);
        a2.w = __shfl_xor_sync(FULL, acc[v].w, off);
        if constexpr (QF) {
          lc2 = __shfl_xor_sync(FULL, lc[v], off);
          u2.x = __shfl_xor_sync(FULL, accu[v].x, off);
          u2.y = __shfl_xor_sync(FULL, accu[v].y, off);
          u2.z = __shfl_xor_sync(FULL, accu[v].z, off);
          u2.w = __shfl_xor_sync(FULL, accu[v].w, off);
        }
        if (g & (off / L::LANES)) {  // canonical order: the lower group's state goes first
          float mt = m2, lt = l2, lct = lc2;
          float4 at = a2, ut = u2;
          if constexpr (QF)
            merge_softmax_q(mt, lt, at, lct, ut, m[v], l[v], acc[v], lc[v], accu[v]);
          else
            merge_softmax(mt, lt, at, m[v], l[v], acc[v]);
          m[v] = mt;
          l[v] = lt;
          acc[v] = at;
          lc[v] = lct;
          accu[v] = ut;
        } else {
          if constexpr (QF)
            merge_softmax_q(m[v], l[v], acc[v], lc[v], accu[v], m2, l2, a2, lc2, u2);
          else
            merge_softmax(m[v], l[v], acc[v], m2, l2, a2);
        }
      }
    }
    if (g != 0) continue;
    if (slot >= 0) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        const int c = L::col(v, q);
        st4(o.pacc + slot * K + c, acc[v]);
        if constexpr (QF) st4(o.pu + slot * K + c, accu[v]);
        if ((c % L::D) == 0) {
          o.pm[slot * NH + c / L::D] = m[v];
          o.pl[slot * NH + c / L::D] = l[v];
          if constexpr (QF) o.pc[slot * NH + c / L::D] = lc[v];
        }
      }
    } else {
      fwd_finish<K, NH>(row, m, l, acc, q, act, o);
      if constexpr (QF) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) {
          const float inv = l[v] > 0.f ? 1.f / l[v] : 0.f, r = l[v] > 0.f ? lc[v] / l[v] : 0.f;
          st4(o.Q + row * K + L::col(v, q), mul4(inv, fma4(-r, acc[v], accu[v])));
        }
      }
    }
  }
}

// heavy rows: fold chunk partials in ascending chunk order (with o.Q: the factored
// backward's u and C partials too, rescaled by the same factors)
template <int K, int NH>
__global__ void __launch_bounds__(kSparseThreads)
gat_fwd_merge_kernel(Items it, int act, FwdOut o) {
  using L = RowLayout<K, NH>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t h = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; h < it.n_heavy; h += nw) {
    const int64_t row = it.heavy_rows[h];
    float m[L::VPL], l[L::VPL], lc[L::VPL];
    float4 acc[L::VPL], accu[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      m[v] = NEG_INF;
      l[v] = lc[v] = 0.f;
      acc[v] = accu[v] = f4(0.f);
    }
    for (int64_t s = it.heavy_off[h]; s < it.heavy_off[h + 1]; ++s) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        const int c = L::col(v, q), hh = c / L::D;
        const float m2 = o.pm[s * NH + hh];
        const float mn = fmaxf(m[v], m2);
        if (mn == NEG_INF) continue;
        const float x = ex2(m[v] - mn), y = ex2(m2 - mn);
        const float4 a2 = ldg4(o.pacc + s * K + c);
        l[v] = fmaf(l[v], x, o.pl[s * NH + hh] * y);
        acc[v] = make_float4(fmaf(acc[v].x, x, a2.x * y), fmaf(acc[v].y, x, a2.y * y),
                             fmaf(acc[v].z, x, a2.z * y), fmaf(acc[v].w, x, a2.w * y));
        if (o.Q) {
          const float4 u2 = ldg4(o.pu + s * K + c);
          lc[v] = fmaf(lc[v], x, o.pc[s * NH + hh] * y);
          accu[v] = make_float4(fmaf(accu[v].x, x, u2.x * y), fmaf(accu[v].y, x, u2.y * y),
                                fmaf(accu[v].z, x, u2.z * y), fmaf(accu[v].w, x, u2.w * y));
        }
        m[v] = mn;
      }
    }
    if (g != 0) continue;
    fwd_finish<K, NH>(row, m, l, acc, q, act, o);
    if (o.Q) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        const float inv = l[v] > 0.f ? 1.f / l[v] : 0.f, r = l[v] > 0.f ? lc[v] / l[v] : 0.f;
        st4(o.Q + row * K + L::col(v, q), mul4(inv, fma4(-r, acc[v], accu[v])));
      }
    }
  }
}

// ---------------------------------------------------------------- backward
using BwdArgs = GatBwdArgs;

template <int K, int NH>
__device__ __forceinline__ void bwd_finish(const BwdArgs& A, int64_t row, int64_t grow, int q,
                                           const float (&ds)[RowLayout<K, NH>::VPL],
                                           const float (&dt)[RowLayout<K, NH>::VPL],
                                           const float4 (&acc)[RowLayout<K, NH>::VPL],
                                           float4 (&da1)[RowLayout<K, NH>::VPL],
                                           float4 (&da2)[RowLayout<K, NH>::VPL]) {
  using L = RowLayout<K, NH>;
#pragma unroll
  for (int v = 0; v < L::VPL; ++v) {
    const int c = L::col(v, q), h = c / L::D, cc = c % L::D;
    const float4 a1 = ldg4(A.a + h * 2 * L::D + cc), a2 = ldg4(A.a + h * 2 * L::D + L::D + cc);
    float4 dp = fma4(ds[v], a1, acc[v]);
    dp = fma4(dt[v], a2, dp);
    st4(A.dP + row * K + c, dp);
    const float4 pj = A.P16 ? ldg4(A.P16 + grow * K + c) : ldg4(A.P + grow * K + c);
    da1[v] = fma4(ds[v], pj, da1[v]);
    da2[v] = fma4(dt[v], pj, da2[v]);
    if (A.ds_out && cc == 0) {
      A.ds_out[row * NH + h] = ds[v];
      A.dt_out[row * NH + h] = dt[v];
    }
  }
}

// ROLE: 0 = both roles over the symmetric CSR; 1 = row role only (CSR pass of a
// directed pattern, ds -> A.ds_dir); 2 = column role only (CSC pass: items are
// columns j, it.col lists the rows i with stored (i,j); ds comes from A.ds_dir)
template <int K, int NH, int U, int ROLE = 0>
__global__ void __launch_bounds__(kSparseThreads)
gat_bwd_kernel(Items it, BwdArgs A) {
  constexpr bool RR = ROLE != 2, CR = ROLE != 1;
  using L = RowLayout<K, NH>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const float slope = A.slope;
  float4 da1[L::VPL], da2[L::VPL];
#pragma unroll
  for (int v = 0; v < L::VPL; ++v) da1[v] = da2[v] = f4(0.f);

  for (int64_t w = gw; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_range<K, NH>(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float4 Pj[L::VPL], Gj[L::VPL], rj[L::VPL], acc[L::VPL];
    float tj[L::VPL], ds[L::VPL], dt[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const int c = L::col(v, q), h = c / L::D;
      Pj[v] = ldg4(A.P + grow * K + c);
      Gj[v] = ldg4(A.G + grow * K + c);
      rj[v] = __ldg(A.rec + grow * NH + h);
      tj[v] = __ldg(A.st + grow * (2 * NH) + NH + h);
      acc[v] = f4(0.f);
      ds[v] = dt[v] = 0.f;
    }
    for (int64_t e0 = beg; e0 < end; e0 += 32) {
      const int cnt = (int)(end - e0 < 32 ? end - e0 : 32);
      const int myc = lane < cnt ? __ldg(it.col + e0 + lane) : 0;
      for (int b = 0; b < cnt; b += L::GROUPS * U) {
        float4 Pi[U][L::VPL], Gi[U][L::VPL], ri[U][L::VPL];
        float ti[U][L::VPL];
        bool val[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int se = b + u * L::GROUPS + g;
          val[u] = se < cnt;
          const int64_t i = __shfl_sync(FULL, myc, se & 31);
#pragma unroll
          for (int v = 0; v < L::VPL; ++v) {
            const int c = L::col(v, q), h = c / L::D;
            if (val[u]) {
              Pi[u][v] = RR ? ldg4(A.P + i * K + c) : f4(0.f);
              Gi[u][v] = CR ? ldg4(A.G + i * K + c) : f4(0.f);
              ri[u][v] = CR ? __ldg(A.rec + i * NH + h) : f4(0.f);
              ti[u][v] = RR ? __ldg(A.st + i * (2 * NH) + NH + h) : 0.f;
            } else {
              Pi[u][v] = Gi[u][v] = ri[u][v] = f4(0.f);
              ti[u][v] = 0.f;
            }
          }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          float d1[L::VPL], d2[L::VPL];
#pragma unroll
          for (int v = 0; v < L::VPL; ++v) {
            d1[v] = dot4(Gj[v], Pi[u][v]);   // G_j . P_i  (row role, dalpha_ji)
            d2[v] = dot4(Gi[u][v], Pj[v]);   // G_i . P_j  (column role, dalpha_ij)
          }
          if (RR) L::head_reduce(d1);
          if (CR) L::head_reduce(d2);
          if (val[u]) {
#pragma unroll
            for (int v = 0; v < L::VPL; ++v) {
              if (RR) {  // row role: entry (j,i) of row j, centre j
                const float pre = rj[v].x + ti[u][v];
                const float e = pre > 0.f ? pre : slope * pre;
                const float aji = ex2(e - rj[v].y) * rj[v].z;
                ds[v] = fmaf(aji * (pre > 0.f ? 1.f : slope), d1[v] - rj[v].w, ds[v]);
              }
              if (CR) {  // column role: entry (i,j) of row i, centre i
                const float pre2 = ri[u][v].x + tj[v];
                const float e2 = pre2 > 0.f ? pre2 : slope * pre2;
                const float aij = ex2(e2 - ri[u][v].y) * ri[u][v].z;
                dt[v] = fmaf(aij * (pre2 > 0.f ? 1.f : slope), d2[v] - ri[u][v].w, dt[v]);
                acc[v] = fma4(aij, Gi[u][v], acc[v]);
              }
            }
          }
        }
      }
    }
#pragma unroll
    for (int off = L::LANES; off < 32; off <<= 1) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        ds[v] += __shfl_xor_sync(FULL, ds[v], off);
        dt[v] += __shfl_xor_sync(FULL, dt[v], off);
        acc[v].x += __shfl_xor_sync(FULL, acc[v].x, off);
        acc[v].y += __shfl_xor_sync(FULL, acc[v].y, off);
        acc[v].z += __shfl_xor_sync(FULL, acc[v].z, off);
        acc[v].w += __shfl_xor_sync(FULL, acc[v].w, off);
      }
    }
    if (g != 0) continue;
    if (slot >= 0) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        const int c = L::col(v, q);
        if (CR) st4(A.pacc + slot * K + c, acc[v]);
        if ((c % L::D) == 0) {
          if (RR) A.pds[slot * NH + c / L::D] = ds[v];
          if (CR) A.pdt[slot * NH + c / L::D] = dt[v];
        }
      }
    } else if (ROLE == 1) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        const int c = L::col(v, q);
        if ((c % L::D) == 0) A.ds_dir[row * NH + c / L::D] = ds[v];
      }
    } else {
      if (ROLE == 2) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) ds[v] = A.ds_dir[row * NH + L::col(v, q) / L::D];
      }
      bwd_finish<K, NH>(A, row, grow, q, ds, dt, acc, da1, da2);
    }
  }
  if (g == 0 && ROLE != 1) {
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const int c = L::col(v, q);
      st4(A.da_part + gw * 2 * K + c, da1[v]);
      st4(A.da_part + gw * 2 * K + K + c, da2[v]);
    }
  }
}

template <int K, int NH, int ROLE = 0>
__global__ void __launch_bounds__(kSparseThreads)
gat_bwd_merge_kernel(Items it, BwdArgs A, int64_t da_row0) {
  using L = RowLayout<K, NH>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  float4 da1[L::VPL], da2[L::VPL];
#pragma unroll
  for (int v = 0; v < L::VPL; ++v) da1[v] = da2[v] = f4(0.f);
  if (g == 0) {
    for (int64_t h = gw; h < it.n_heavy; h += nw) {
      const int64_t row = it.heavy_rows[h], grow = it.row_begin + row;
      float ds[L::VPL], dt[L::VPL];
      float4 acc[L::VPL];
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        ds[v] = dt[v] = 0.f;
        acc[v] = f4(0.f);
      }
      for (int64_t s = it.heavy_off[h]; s < it.heavy_off[h + 1]; ++s) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) {
          const int c = L::col(v, q), hh = c / L::D;
          if (ROLE != 1) acc[v] = add4(acc[v], ldg4(A.pacc + s * K + c));
          if (ROLE != 2) ds[v] += A.pds[s * NH + hh];
          if (ROLE != 1) dt[v] += A.pdt[s * NH + hh];
        }
      }
      if (ROLE == 1) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) {
          const int c = L::col(v, q);
          if ((c % L::D) == 0) A.ds_dir[row * NH + c / L::D] = ds[v];
        }
        continue;
      }
      if (ROLE == 2) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) ds[v] = A.ds_dir[row * NH + L::col(v, q) / L::D];
      }
      bwd_finish<K, NH>(A, row, grow, q, ds, dt, acc, da1, da2);
    }
#pragma unroll
    for (int v = 0; v < L::VPL && ROLE != 1; ++v) {
      const int c = L::col(v, q);
      st4(A.da_part + (da_row0 + gw) * 2 * K + c, da1[v]);
      st4(A.da_part + (da_row0 + gw) * 2 * K + K + c, da2[v]);
    }
  }
}

// G = dH_out (.) sigma'(Z) ; rec = {s, m, 1/l, delta = G^h . Z^h} (per head).
// TG = bf16 (BF16 mode, reading B1): G is rounded to bfloat16 first and the rounded
// G~ is what delta uses and what is stored.
template <int K, int NH, typename TG = float>
__global__ void __launch_bounds__(kSparseThreads)
gat_bwd_prologue_kernel(int64_t n_local, int64_t row_begin, const float* __restrict__ dHout,
                        const float* __restrict__ Z, const float* __restrict__ st,
                        const float* __restrict__ mrow, const float* __restrict__ lrow, int act,
                        TG* __restrict__ G, float4* __restrict__ rec, PeerRows peers,
                        const float* __restrict__ Q, float* __restrict__ ds_row) {
  using L = RowLayout<K, NH>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t slots = (n_local + L::GROUPS - 1) / L::GROUPS;
  for (int64_t rs = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; rs < slots; rs += nw) {
    const int64_t row = rs * L::GROUPS + g;
    const bool ok = row < n_local;
    float dl[L::VPL], dq[L::VPL];
    float4 gv[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const int c = L::col(v, q);
      float4 z = f4(0.f), dh = f4(0.f), qv = f4(0.f);
      if (ok) {
        z = ldg4(Z + row * K + c);
        dh = ldg4(dHout + row * K + c);
        if (Q) qv = ldg4(Q + row * K + c);
      }
      gv[v] = make_float4(dh.x * act_grad(act, z.x), dh.y * act_grad(act, z.y),
                          dh.z * act_grad(act, z.z), dh.w * act_grad(act, z.w));
      if constexpr (sizeof(TG) == 2) gv[v] = round_bf4(gv[v]);
      dl[v] = dot4(gv[v], z);
      dq[v] = dot4(gv[v], qv);  // factored backward: ds_j = G_j . Q_j (gat_args.cuh)
    }
    L::head_reduce(dl);
    if (Q) L::head_reduce(dq);
    if (!ok) continue;
    const int64_t grow = row_begin + row;
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const int c = L::col(v, q), h = c / L::D;
      st4(G + grow * K + c, gv[v]);
      const uint32_t pm = peers.n ? peers.mask[row] : 0u;
      for (int pi = 0; pi < peers.n; ++pi)  // the peers whose rows reference this one
        if ((pm >> pi) & 1u) st4(reinterpret_cast<TG*>(peers.a[pi]) + grow * K + c, gv[v]);
      if ((c % L::D) == 0) {
        const float lv = lrow[row * NH + h];
        const float4 r4 = make_float4(st[grow * 2 * NH + h], mrow[row * NH + h],
                                      lv > 0.f ? 1.f / lv : 0.f, dl[v]);
        rec[grow * NH + h] = r4;
        for (int pi = 0; pi < peers.n; ++pi)
          if ((pm >> pi) & 1u) reinterpret_cast<float4*>(peers.b[pi])[grow * NH + h] = r4;
        if (Q) ds_row[row * NH + h] = dq[v];
      }
    }
  }
}

// da[h][0:D] = sum_w part[w][c], da[h][D:2D] = sum_w part[w][K + c]   (fixed order)
__global__ void __launch_bounds__(1024)
gat_da_reduce_kernel(const float* __restrict__ part, int64_t rows, int K, int D,
                     float* __restrict__ da) {
  // block: 32 columns x 32 row-lanes; each row-lane sums a strided subset, then a
  // fixed-order tree over the row-lanes (deterministic)
  __shared__ float red[32][33];
  const int tx = threadIdx.x & 31, ty = threadIdx.x >> 5;
  const int c2 = blockIdx.x * 32 + tx;
  float s = 0.f;
  if (c2 < 2 * K) {
#pragma unroll 8
    for (int64_t r = ty; r < rows; r += 32) s += part[r * 2 * K + c2];
  }
  red[ty][tx] = s;
  __syncthreads();
  for (int o = 16; o > 0; o >>= 1) {
    if (ty < o) red[ty][tx] += red[ty + o][tx];
    __syncthreads();
  }
  if (ty == 0 && c2 < 2 * K) {
    const int c = c2 % K, h = c / D, cc = c % D;
    da[h * 2 * D + (c2 >= K ? D : 0) + cc] = red[0][tx];
  }
}

// W_ext = [W | log2e W a1^h ... | log2e W a2^h ...]   (a' = W a, Table 2).
// The scores s, t (and the saved row maxima m) are stored in log2 units so every
// exponential is a single ex2; LReLU commutes with the positive scale.
__global__ void gat_wext_kernel(const float* __restrict__ W, const float* __restrict__ a, int k_in,
                                int K, int NH, int NE, float* __restrict__ WextT) {
  const int D = K / NH;
  for (int idx = blockIdx.x * blockDim.x + threadIdx.x; idx < k_in * NE;
       idx += gridDim.x * blockDim.x) {
    const int c = idx / k_in, r = idx % k_in;  // output [NE x k_in] (B given as [N x K])
    float v;
    if (c < K) {
      v = W[r * K + c];
    } else if (c >= K + 2 * NH) {
      v = 0.f;  // padding column (N multiple of 4)
    } else {
      const int h = (c - K) % NH, which = (c - K) / NH;
      v = 0.f;
      for (int x = 0; x < D; ++x) v = fmaf(W[r * K + h * D + x], a[h * 2 * D + which * D + x], v);
      v *= kLog2e;  // scores are kept in log2 units: e2 = LReLU(s2 + t2) = log2(e) * e_nat
    }
    WextT[idx] = v;
  }
}

// alpha of sampled stored entries, recomputed from saved statistics
__global__ void gat_debug_alpha_kernel(const int64_t* __restrict__ rp, int64_t n_local,
                                       const int32_t* __restrict__ col, int64_t row_begin,
                                       const float* __restrict__ st, const float* __restrict__ mrow,
                                       const float* __restrict__ lrow, int NH, float slope,
                                       const int64_t* __restrict__ pos, int64_t count,
                                       float* __restrict__ out) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= count * NH) return;
  const int64_t e = pos[t / NH];
  const int h = (int)(t % NH);
  int64_t lo = 0, hi = n_local;  // last row with rp[row] <= e
  while (hi - lo > 1) {
    const int64_t mid = (lo + hi) / 2;
    if (rp[mid] <= e) lo = mid; else hi = mid;
  }
  const int64_t j = col[e];
  const float pre = st[(row_begin + lo) * 2 * NH + h] + st[j * 2 * NH + NH + h];
  const float x = pre > 0.f ? pre : slope * pre;
  out[t] = exp2f(x - mrow[lo * NH + h]) / lrow[lo * NH + h];
}

// ---------------------------------------------------------------- layout
// the factored backward (gat_args.cuh): symmetric patterns run the k' = 128
// kernels or the generic ones (forward with QF, backward = the column-role pass
// over the CSR, which for a symmetric pattern lists every column's entries);
// directed patterns skip their row pass (column pass over the CSC only)
// Plan option gat_factored: 1 (default) = k' = 128 only; 2 = every width; 0 = never.
// Measured: k' = 128 at C5 1.45x faster step; k' = 64 at C2 (L2-resident, so the
// gathered bytes it saves cost nothing) 0.81 -> 0.87 ms, hence k' = 128 only by default.
bool factored(const Plan& p, const GatShape& g) {
  const int mode = p.gat_factored;
  return mode > 0 && (mode == 2 || gat_k128_supported(g.k_out, g.heads));
}

struct SavedGat {
  float *P, *st, *Z, *m, *l;
  bf16* P16;  // BF16 mode: P stored as bfloat16 (P == NULL)
  float* Q;   // factored backward: [n_local x K] (NULL otherwise)
};
SavedGat carve_saved(const Plan& p, const GatShape& g, void* base) {
  Carver c(base);
  SavedGat s;
  s.P = nullptr;
  s.P16 = nullptr;
  if (g.bf16)
    s.P16 = c.take<bf16>((size_t)p.n * g.k_out);
  else
    s.P = c.take<float>((size_t)p.n * g.k_out);
  s.st = c.take<float>((size_t)p.n * 2 * g.heads);
  s.Z = c.take<float>((size_t)p.n_local * g.k_out);
  s.m = c.take<float>((size_t)p.n_local * g.heads);
  s.l = c.take<float>((size_t)p.n_local * g.heads);
  s.Q = factored(p, g) ? c.take<float>((size_t)p.n_local * g.k_out) : nullptr;
  return s;
}
size_t saved_size(const Plan& p, const GatShape& g) {
  Carver c(nullptr);
  if (g.bf16)
    c.take<bf16>((size_t)p.n * g.k_out);
  else
    c.take<float>((size_t)p.n * g.k_out);
  c.take<float>((size_t)p.n * 2 * g.heads);
  c.take<float>((size_t)p.n_local * g.k_out);
  c.take<float>((size_t)p.n_local * g.heads);
  c.take<float>((size_t)p.n_local * g.heads);
  if (factored(p, g)) c.take<float>((size_t)p.n_local * g.k_out);
  return c.off + 256;
}

struct WsGat {
  float *Wext, *pacc, *pm, *pl, *G, *dP, *da_part, *gemm, *ds_dir, *ds_row;
  bf16* G16;  // BF16 mode: G stored as bfloat16 (G == NULL)
  float4* rec;
  void* saved_inf;  // saved-layout scratch for inference
};
int64_t da_rows() { return (int64_t)kMaxSparseBlocks * (kSparseThreads / 32) * 3; }

WsGat carve_ws(const Plan& p, const GatShape& g, void* base, size_t* total) {
  Carver c(base);
  WsGat w;
  const int NE = (g.k_out + 2 * g.heads + 3) / 4 * 4;
  // replicated (n-row) arrays first: their offsets are the same on every rank, which
  // the peer-memory exchange relies on (agnn_plan_register maps whole buffers)
  w.G = nullptr;
  w.G16 = nullptr;
  if (g.bf16)
    w.G16 = c.take<bf16>((size_t)p.n * g.k_out);
  else
    w.G = c.take<float>((size_t)p.n * g.k_out);
  w.rec = c.take<float4>((size_t)p.n * g.heads);
  w.saved_inf = c.take<char>(saved_size(p, g));  // its replicated prefix (P, st) too
  w.Wext = c.take<float>((size_t)g.k_in * NE);
  w.pacc = c.take<float>((size_t)p.max_chunks() * 3 * g.k_out);
  w.pm = c.take<float>((size_t)p.max_chunks() * g.heads);
  w.pl = c.take<float>((size_t)p.max_chunks() * g.heads);
  w.ds_dir = c.take<float>(p.csc_ptr ? (size_t)p.n_local * g.heads : 0);
  w.ds_row = c.take<float>(factored(p, g) ? (size_t)p.n_local * g.heads : 0);
  w.dP = c.take<float>((size_t)p.n_local * g.k_out);
  w.da_part = c.take<float>((size_t)da_rows() * 2 * g.k_out);
  w.gemm = c.take<float>(gemm_tn_ws_floats(g.k_in, g.k_out));
  if (total) *total = c.off + 256;
  return w;
}

}  // namespace

size_t gat_saved_bytes(const Plan& p, const GatShape& g) { return saved_size(p, g); }
size_t gat_workspace_bytes(const Plan& p, const GatShape& g) {
  size_t t = 0;
  carve_ws(p, g, nullptr, &t);
  return t;
}

// ---------------------------------------------------------------- dispatch
#define AGNN_GAT_DISPATCH(K_, NH_, CALL)                                                  \
  do {                                                                                    \
    bool _done = false;                                                                   \
    AGNN_GAT_CASE(16, 1, CALL) AGNN_GAT_CASE(16, 2, CALL) AGNN_GAT_CASE(16, 4, CALL)      \
    AGNN_GAT_CASE(32, 1, CALL) AGNN_GAT_CASE(32, 2, CALL) AGNN_GAT_CASE(32, 4, CALL)      \
    AGNN_GAT_CASE(32, 8, CALL) AGNN_GAT_CASE(64, 1, CALL) AGNN_GAT_CASE(64, 2, CALL)      \
    AGNN_GAT_CASE(64, 4, CALL) AGNN_GAT_CASE(64, 8, CALL) AGNN_GAT_CASE(128, 1, CALL)     \
    AGNN_GAT_CASE(128, 2, CALL) AGNN_GAT_CASE(128, 4, CALL) AGNN_GAT_CASE(128, 8, CALL)   \
    AGNN_GAT_CASE(256, 1, CALL) AGNN_GAT_CASE(256, 2, CALL) AGNN_GAT_CASE(256, 4, CALL)   \
    AGNN_GAT_CASE(256, 8, CALL)                                                           \
    if (!_done) return fail(AGNN_EUNSUPPORTED, "GAT: unsupported (k_out, heads)");        \
  } while (0)
#define AGNN_GAT_CASE(KK, HH, CALL)                       \
  if (!_done && K_ == KK && NH_ == HH) {                  \
    constexpr int K = KK, NH = HH;                        \
    CALL;                                                 \
    _done = true;                                         \
  }

template <int K>
constexpr int fwd_unroll() { return K >= 256 ? 2 : 4; }
template <int K>
constexpr int bwd_unroll() { return K >= 256 ? 1 : (K >= 128 ? 2 : 4); }

agnn_status gat_forward(const Plan& p, const GatShape& g, const float* W, const float* a,
                        const float* H_in, float* H_out, void* saved, void* ws, cudaStream_t s) {
  WsGat w = carve_ws(p, g, ws, nullptr);
  SavedGat sv = carve_saved(p, g, saved ? saved : w.saved_inf);
  const int K_ = g.k_out, NH_ = g.heads, NEs = g.k_out + 2 * g.heads, NE = (NEs + 3) / 4 * 4;
  gat_wext_kernel<<<64, 256, 0, s>>>(W, a, g.k_in, g.k_out, g.heads, NE, w.Wext);
  AGNN_LAUNCH_CHECK("gat_wext_kernel");
  // P (and s, t) for the local rows, written at their global offsets
  float* stloc = sv.st + p.row_begin * 2 * g.heads;
  agnn_status st;
  if (g.bf16) {
    // BF16 mode (reading B1): the tcgen05 epilogue rounds P to bfloat16; s, t come
    // from the same (unrounded) accumulators; then the plain all-gather of P~ | st
    Items it = items_of(p);
    FwdOut o{saved ? sv.Z : nullptr, H_out, saved ? sv.m : nullptr, saved ? sv.l : nullptr,
             w.pacc, w.pm, w.pl, saved ? sv.Q : nullptr, w.pacc + p.max_chunks() * g.k_out,
             w.pacc + 2 * p.max_chunks() * g.k_out};
    if ((st = gemm_rows_bf16(H_in, p.n_local, g.k_in, w.Wext, NEs, sv.P16 + p.row_begin * g.k_out,
                             g.k_out, stloc, w.dP, s)) != AGNN_OK)
      return st;
    if (p.world > 1) {
      const RowArray ra[2] = {{reinterpret_cast<float*>(sv.P16), g.k_out / 2}, {sv.st, 2 * g.heads}};
      if ((st = allgather_rows(p, ra, 2, s)) != AGNN_OK) return st;
    }
    // gathered per edge: a bf16 row of P and the t_j of the heads
    const Items ith = l2_hinted(it, p, 2 * (int64_t)g.k_out + 4 * g.heads);
    if ((st = gat_fwd_k128_bf16(ith, g.heads, sv.P16, sv.st, g.slope, g.act, o, s)) != AGNN_OK)
      return st;
    if (it.n_heavy > 0) {
      AGNN_GAT_DISPATCH(K_, NH_, (gat_fwd_merge_kernel<K, NH>
                                  <<<kNumSMs * 2, kSparseThreads, 0, s>>>(it, g.act, o)));
      AGNN_LAUNCH_CHECK("gat_fwd_merge_kernel");
    }
    return AGNN_OK;
  }
  // P | s t for the local rows, written at their global offsets.  With P > 1 over peer
  // memory the GEMM epilogue also stores every row into the replicas of the peers whose
  // CSR references it (fused GEMM -> needed-rows exchange, NVLink stores overlapping
  // the next tiles), between an entry and an exit barrier; otherwise the rows are
  // pushed after the GEMM (comm.cu)
  float* Ploc = sv.P + p.row_begin * g.k_out;
  PeerOut po;
  const bool fuse = p.world > 1 && peer_out(p, Ploc, stloc, po);
  if (fuse && (st = peer_barrier(p, s)) != AGNN_OK) return st;
  bool fused = false;
  if ((st = gemm_rows(H_in, p.n_local, g.k_in, w.Wext, true, NE, Ploc, g.k_out, stloc, s,
                      nullptr, 0, NEs, fuse ? &po : nullptr, &fused)) != AGNN_OK)
    return st;
  if (fused) {
    if ((st = peer_barrier(p, s)) != AGNN_OK) return st;
  } else if (p.world > 1) {
    if (fuse && (st = peer_barrier(p, s)) != AGNN_OK) return st;  // (same barrier count)
    const RowArray ra[2] = {{sv.P, g.k_out}, {sv.st, 2 * g.heads}};
    if ((st = allgather_rows(p, ra, 2, s)) != AGNN_OK) return st;
  }
  Items it = items_of(p);
  FwdOut o{saved ? sv.Z : nullptr, H_out, saved ? sv.m : nullptr, saved ? sv.l : nullptr,
           w.pacc, w.pm, w.pl, saved ? sv.Q : nullptr, w.pacc + p.max_chunks() * g.k_out,
           w.pacc + 2 * p.max_chunks() * g.k_out};
  if (gat_k128_supported(g.k_out, g.heads)) {
    const Items ith = l2_hinted(it, p, 4 * (int64_t)g.k_out + 4 * g.heads);
    if ((st = gat_fwd_k128(ith, g.heads, sv.P, sv.st, g.slope, g.act, o, s)) != AGNN_OK)
      return st;
  } else if (it.n_chunks + it.n_light > 0) {
    if (o.Q)
      AGNN_GAT_DISPATCH(K_, NH_, (gat_fwd_kernel<K, NH, fwd_unroll<K>(), true>
                                  <<<grid_of(gat_fwd_kernel<K, NH, fwd_unroll<K>(), true>),
                                     kSparseThreads, 0, s>>>(it, sv.P, sv.st, g.slope, g.act, o)));
    else
      AGNN_GAT_DISPATCH(K_, NH_, (gat_fwd_kernel<K, NH, fwd_unroll<K>(), false>
                                  <<<grid_of(gat_fwd_kernel<K, NH, fwd_unroll<K>(), false>),
                                     kSparseThreads, 0, s>>>(it, sv.P, sv.st, g.slope, g.act, o)));
    AGNN_LAUNCH_CHECK("gat_fwd_kernel");
  }
  if (it.n_heavy > 0) {
    AGNN_GAT_DISPATCH(K_, NH_, (gat_fwd_merge_kernel<K, NH>
                                <<<kNumSMs * 2, kSparseThreads, 0, s>>>(it, g.act, o)));
    AGNN_LAUNCH_CHECK("gat_fwd_merge_kernel");
  }
  return AGNN_OK;
}

agnn_status gat_backward(const Plan& p, const GatShape& g, const float* W, const float* a,
                         const float* H_in, const void* saved, const float* dH_out,
                         float* dH_in, float* dW, float* da, void* ws, cudaStream_t s) {
  if (!saved) return fail(AGNN_EINVAL, "agnn_backward: saved == NULL");
  const bool directed = p.directed();
  if (directed && !p.csc_ptr)
    return fail(AGNN_EUNSUPPORTED,
                "agnn_backward: a directed pattern needs world == 1 and every row in the plan");
  WsGat w = carve_ws(p, g, ws, nullptr);
  SavedGat sv = carve_saved(p, g, const_cast<void*>(saved));
  const int K_ = g.k_out, NH_ = g.heads;
  Items it = items_of(p);
  agnn_status st;
  // peer memory: the prologue stores G | rec also into the replicas of the peers whose
  // CSR references the row (fused prologue -> needed-rows exchange)
  PeerRows pr;
  const bool fuse_g = p.world > 1 && peer_rows(p, g.bf16 ? (void*)w.G16 : (void*)w.G, w.rec, pr);
  if (fuse_g && (st = peer_barrier(p, s)) != AGNN_OK) return st;
  if (g.bf16) {
    if (directed)
      return fail(AGNN_EUNSUPPORTED, "AGNN_PREC_BF16: symmetric patterns only");
    AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_prologue_kernel<K, NH, bf16>
                                <<<grid_of(gat_bwd_prologue_kernel<K, NH, bf16>), kSparseThreads, 0,
                                   s>>>(p.n_local, p.row_begin, dH_out, sv.Z, sv.st, sv.m, sv.l,
                                        g.act, w.G16, w.rec, pr, sv.Q, w.ds_row)));
  } else {
    AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_prologue_kernel<K, NH>
                                <<<grid_of(gat_bwd_prologue_kernel<K, NH>), kSparseThreads, 0, s>>>(
                                    p.n_local, p.row_begin, dH_out, sv.Z, sv.st, sv.m, sv.l, g.act,
                                    w.G, w.rec, pr, sv.Q, w.ds_row)));
  }
  AGNN_LAUNCH_CHECK("gat_bwd_prologue_kernel");
  if (fuse_g) {  // exit barrier: the prologue's peer stores are visible
    if ((st = peer_barrier(p, s)) != AGNN_OK) return st;
  } else if (p.world > 1) {  // NCCL: G | rec blocks -> every replica
    const RowArray ra[2] = {{g.bf16 ? reinterpret_cast<float*>(w.G16) : w.G,
                             g.bf16 ? g.k_out / 2 : g.k_out},
                            {reinterpret_cast<float*>(w.rec), 4 * g.heads}};
    if ((st = allgather_rows(p, ra, 2, s)) != AGNN_OK) return st;
  }
  BwdArgs A{sv.P, sv.st, w.G, w.rec, a, g.slope, w.dP, w.pacc, w.pm, w.pl, w.da_part,
            nullptr, nullptr, w.ds_dir, sv.P16, w.G16, w.ds_row};
  int64_t main_warps = 0, merge_warps = 0;
  bool merged = false;  // the branch below ran its own heavy-row merge
  if (directed) {
    // row role over the CSR (ds_j), then the column role over the CSC (dt_j, acc_j, dP_j);
    // factored (Q saved by the forward): ds_j = G_j . Q_j from the prologue replaces
    // the whole row pass (the forward visited exactly row j's entries)
    Items itc = items_of_csc(p);
    if (sv.Q) {
      A.ds_dir = w.ds_row;
    } else {
      AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_kernel<K, NH, bwd_unroll<K>(), 1>
                                  <<<grid_of(gat_bwd_kernel<K, NH, bwd_unroll<K>(), 1>),
                                     kSparseThreads, 0, s>>>(it, A)));
      AGNN_LAUNCH_CHECK("gat_bwd_row_kernel");
      if (it.n_heavy > 0) {
        AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_merge_kernel<K, NH, 1>
                                    <<<kNumSMs * 2, kSparseThreads, 0, s>>>(it, A, 0)));
        AGNN_LAUNCH_CHECK("gat_bwd_merge_kernel");
      }
    }
    it = itc;
    AGNN_GAT_DISPATCH(K_, NH_, (main_warps = (int64_t)grid_of(gat_bwd_kernel<K, NH, bwd_unroll<K>(), 2>) *
                                             (kSparseThreads / 32)));
    AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_kernel<K, NH, bwd_unroll<K>(), 2>
                                <<<(unsigned)(main_warps / 8), kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("gat_bwd_col_kernel");
    AGNN_GAT_DISPATCH(K_, NH_, (merge_warps = (int64_t)grid_of(gat_bwd_merge_kernel<K, NH, 2>) *
                                              (kSparseThreads / 32)));
    AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_merge_kernel<K, NH, 2>
                                <<<(unsigned)(merge_warps / 8), kSparseThreads, 0, s>>>(
                                    it, A, main_warps)));
    AGNN_LAUNCH_CHECK("gat_bwd_merge_kernel");
  } else if (sv.Q && gat_k128_supported(g.k_out, g.heads)) {
    // factored: gathered per edge only G_i and the records rec_i of the heads
    const Items ith = l2_hinted(it, p, (g.bf16 ? 2 : 4) * (int64_t)g.k_out + 16 * g.heads);
    if ((st = gat_bwd_k128f(ith, g.heads, A, &main_warps, s)) != AGNN_OK) return st;
  } else if (sv.Q) {
    // factored, generic widths: the column-role pass of the directed backward over the
    // (symmetric) CSR, with ds_j = G_j . Q_j from the prologue in place of the row pass
    merged = true;
    A.ds_dir = w.ds_row;
    AGNN_GAT_DISPATCH(K_, NH_, (main_warps = (int64_t)grid_of(gat_bwd_kernel<K, NH, bwd_unroll<K>(), 2>) *
                                             (kSparseThreads / 32)));
    AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_kernel<K, NH, bwd_unroll<K>(), 2>
                                <<<(unsigned)(main_warps / 8), kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("gat_bwd_kernel");
    AGNN_GAT_DISPATCH(K_, NH_, (merge_warps = (int64_t)grid_of(gat_bwd_merge_kernel<K, NH, 2>) *
                                              (kSparseThreads / 32)));
    AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_merge_kernel<K, NH, 2>
                                <<<(unsigned)(merge_warps / 8), kSparseThreads, 0, s>>>(
                                    it, A, main_warps)));
    AGNN_LAUNCH_CHECK("gat_bwd_merge_kernel");
  } else if (gat_k128_supported(g.k_out, g.heads)) {
    // gathered per edge: rows P_i and G_i, the record rec_i and t_i of the heads
    const Items ith =
        l2_hinted(it, p, 2 * (g.bf16 ? 2 : 4) * (int64_t)g.k_out + 20 * g.heads);
    if ((st = gat_bwd_k128(ith, g.heads, A, &main_warps, s)) != AGNN_OK) return st;
  } else {
    AGNN_GAT_DISPATCH(K_, NH_, (main_warps = (int64_t)grid_of(gat_bwd_kernel<K, NH, bwd_unroll<K>()>) *
                                             (kSparseThreads / 32)));
    AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_kernel<K, NH, bwd_unroll<K>()>
                                <<<(unsigned)(main_warps / 8), kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("gat_bwd_kernel");
  }
  if (!directed && !merged) {
    AGNN_GAT_DISPATCH(K_, NH_, (merge_warps = (int64_t)grid_of(gat_bwd_merge_kernel<K, NH>) *
                                              (kSparseThreads / 32)));
    AGNN_GAT_DISPATCH(K_, NH_, (gat_bwd_merge_kernel<K, NH>
                                <<<(unsigned)(merge_warps / 8), kSparseThreads, 0, s>>>(
                                    it, A, main_warps)));
    AGNN_LAUNCH_CHECK("gat_bwd_merge_kernel");
  }
  const int64_t da_rows_used = main_warps + merge_warps;
  if (da) {
    gat_da_reduce_kernel<<<(2 * g.k_out + 31) / 32, 1024, 0, s>>>(
        w.da_part, da_rows_used, g.k_out, g.k_out / g.heads, da);
    AGNN_LAUNCH_CHECK("gat_da_reduce_kernel");
    if (p.world > 1 && (st = allreduce_sum(p, da, 2 * (int64_t)g.k_out, s)) != AGNN_OK) return st;
  }
  if (dW) {
    if ((st = gemm_tn(H_in, p.n_local, g.k_in, w.dP, g.k_out, dW, w.gemm, s)) != AGNN_OK) return st;
    if (p.world > 1 && (st = allreduce_sum(p, dW, (int64_t)g.k_in * g.k_out, s)) != AGNN_OK)
      return st;
  }
  if (dH_in) {
    if ((st = gemm_rows(w.dP, p.n_local, g.k_out, W, true, g.k_in, dH_in, g.k_in, nullptr, s)) !=
        AGNN_OK)
      return st;
  }
  return AGNN_OK;
}

agnn_status gat_debug_alpha(const Plan& p, const GatShape& g, const void* saved,
                            const int64_t* edge_pos, int64_t count, float* out, cudaStream_t s) {
  if (!saved) return fail(AGNN_EINVAL, "debug_attention: saved == NULL");
  if (count <= 0) return AGNN_OK;
  SavedGat sv = carve_saved(p, g, const_cast<void*>(saved));
  const int64_t tot = count * g.heads;
  gat_debug_alpha_kernel<<<(unsigned)((tot + 255) / 256), 256, 0, s>>>(
      p.row_ptr, p.n_local, p.col_idx, p.row_begin, sv.st, sv.m, sv.l, g.heads, g.slope, edge_pos,
      count, out);
  AGNN_LAUNCH_CHECK("gat_debug_alpha_kernel");
  return AGNN_OK;
}

}  // namespace agnn
