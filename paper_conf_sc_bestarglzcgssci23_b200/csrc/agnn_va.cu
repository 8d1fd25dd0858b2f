// agnn_va.cu — fused sparse kernels of the AGNN and VA layers.
//
// Both models aggregate first (Phi o (+) order freedom):
//   X = Psi H  (fused SDDMM -> [softmax] -> SpMM, one pass over the CSR)
//   Z = X W, H_out = sigma(Z)  (dense GEMM with the activation in its epilogue)
// VA   (Eq. 7 at :262):  S_ij = H_i . H_j,  X_i = sum_j S_ij H_j
// AGNN (reading A8):     c_ij = beta H_i.H_j / (nu_i nu_j),
//      alpha = row softmax(c), X_i = sum_j alpha_ij H_j.  |c_ij| <= |beta| (cosine),
//      so the softmax uses the fixed shift m_i = |beta| (shift invariance; no
//      running max and no rescaling, and chunk partials merge by plain sums).
// Backward (Eq. 6, dPsi/dW = 0; VA Eq. 11-13 at :289-298),
// after G = dH_out (.) sigma'(Z), dW = X^T G, M = G W^T, one pass over the
// symmetric CSR visits every stored entry (j,i) once for both roles:
//   VA   dH_j = sum_i (M_j.H_i + M_i.H_j) H_i + (H_i.H_j) M_i      (N+ H + (A^T (.) H_x) M)
//   AGNN dc_ji = beta alpha_ji (M_j.H_i - delta_j), dc_ij = beta alpha_ij (M_i.H_j - delta_i)
//        dH^_j += (dc_ji + dc_ij) H^_i ; acc_j += alpha_ij M_i
//        dH_j = acc_j + (dH^_j - (dH^_j.H^_j) H^_j) / nu_j
#include "av_args.cuh"

namespace agnn {

namespace {

constexpr unsigned FULL = 0xffffffffu;
enum { VA = AV_VA, AG = AV_AG };



template <int K>
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

template <int K, int MODEL>
__device__ __forceinline__ void fwd_store(const AvFwd& A, int64_t row, int q, float l,
                                          const float4 (&acc)[RowLayout<K, 1>::VPL]) {
  using L = RowLayout<K, 1>;
  const float inv = (MODEL == AG) ? (l > 0.f ? 1.f / l : 0.f) : 1.f;
#pragma unroll
  for (int v = 0; v < L::VPL; ++v) st4(A.X + row * K + L::col(v, q), mul4(inv, acc[v]));
  if (MODEL == AG && q == 0) A.l[row] = l;
}

template <int K, int MODEL, int U>
__global__ void __launch_bounds__(kSparseThreads) av_fwd_kernel(Items it, AvFwd A) {
  using L = RowLayout<K, 1>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const float beta = A.beta, bound = A.bound;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_range<K>(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float4 Hi[L::VPL], acc[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      Hi[v] = ldg4(A.H + grow * K + L::col(v, q));
      acc[v] = f4(0.f);
    }
    const float scale_i = (MODEL == AG) ? beta / __ldg(A.nu + grow) : 1.f;
    float l = 0.f;
    for (int64_t e0 = beg; e0 < end; e0 += 32) {
      const int cnt = (int)(end - e0 < 32 ? end - e0 : 32);
      const int myc = lane < cnt ? __ldg(it.col + e0 + lane) : 0;
      for (int b = 0; b < cnt; b += L::GROUPS * U) {
        float4 Hj[U][L::VPL];
        float nuj[U], d[U][L::VPL];
        bool val[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int se = b + u * L::GROUPS + g;
          val[u] = se < cnt;
          const int64_t j = __shfl_sync(FULL, myc, se & 31);
#pragma unroll
          for (int v = 0; v < L::VPL; ++v)
            Hj[u][v] = val[u] ? ldg4(A.H + j * K + L::col(v, q)) : f4(0.f);
          nuj[u] = (MODEL == AG && val[u]) ? __ldg(A.nu + j) : 1.f;
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
#pragma unroll
          for (int v = 0; v < L::VPL; ++v) d[u][v] = dot4(Hi[v], Hj[u][v]);
          L::head_reduce(d[u]);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (!val[u]) continue;
          float wgt;
          if (MODEL == AG) {
            wgt = ex2((scale_i * d[u][0] / nuj[u] - bound) * kLog2e);   // exp(c_ij - |beta|)
            l += wgt;
          } else {
            wgt = d[u][0];                                              // S_ij = H_i . H_j
          }
#pragma unroll
          for (int v = 0; v < L::VPL; ++v) acc[v] = fma4(wgt, Hj[u][v], acc[v]);
        }
      }
    }
#pragma unroll
    for (int off = L::LANES; off < 32; off <<= 1) {
      l += __shfl_xor_sync(FULL, l, off);
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        acc[v].x += __shfl_xor_sync(FULL, acc[v].x, off);
        acc[v].y += __shfl_xor_sync(FULL, acc[v].y, off);
        acc[v].z += __shfl_xor_sync(FULL, acc[v].z, off);
        acc[v].w += __shfl_xor_sync(FULL, acc[v].w, off);
      }
    }
    if (g != 0) continue;
    if (slot >= 0) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) st4(A.pacc + slot * K + L::col(v, q), acc[v]);
      if (MODEL == AG && q == 0) A.pl[slot] = l;
    } else {
      fwd_store<K, MODEL>(A, row, q, l, acc);
    }
  }
}

template <int K, int MODEL>
__global__ void __launch_bounds__(kSparseThreads) av_fwd_merge_kernel(Items it, AvFwd A) {
  using L = RowLayout<K, 1>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t h = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; h < it.n_heavy; h += nw) {
    const int64_t row = it.heavy_rows[h];
    float4 acc[L::VPL];
    float l = 0.f;
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) acc[v] = f4(0.f);
    for (int64_t s = it.heavy_off[h]; s < it.heavy_off[h + 1]; ++s) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) acc[v] = add4(acc[v], ldg4(A.pacc + s * K + L::col(v, q)));
      if (MODEL == AG) l += A.pl[s];
    }
    if (g == 0) fwd_store<K, MODEL>(A, row, q, l, acc);
  }
}

// nu_i = max(||H_i||, eps)
template <int K>
__global__ void __launch_bounds__(kSparseThreads)
nu_kernel(const float* __restrict__ H, int64_t n_local, float eps, float* __restrict__ nu) {
  using L = RowLayout<K, 1>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t slots = (n_local + L::GROUPS - 1) / L::GROUPS;
  for (int64_t rs = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; rs < slots; rs += nw) {
    const int64_t row = rs * L::GROUPS + g;
    const bool ok = row < n_local;
    float d[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const float4 h = ok ? ldg4(H + row * K + L::col(v, q)) : f4(0.f);
      d[v] = dot4(h, h);
    }
    L::head_reduce(d);
    if (ok && q == 0) nu[row] = fmaxf(sqrtf(d[0]), eps);
  }
}

// BF16 storage (reading B2): H~ = bf16(H) of the local rows into the (replicated) H16
// at their global offsets, and AGNN's nu_i = max(|H~_i|, eps) of the rounded row
template <int K>
__global__ void __launch_bounds__(kSparseThreads)
av_round_kernel(const float* __restrict__ H, int64_t n_local, float eps, bf16* __restrict__ H16,
                float* __restrict__ nu) {
  using L = RowLayout<K, 1>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t slots = (n_local + L::GROUPS - 1) / L::GROUPS;
  for (int64_t rs = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; rs < slots; rs += nw) {
    const int64_t row = rs * L::GROUPS + g;
    const bool ok = row < n_local;
    float d[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      const float4 h = ok ? round_bf4(ldg4(H + row * K + L::col(v, q))) : f4(0.f);
      if (ok) st4(H16 + row * K + L::col(v, q), h);
      d[v] = dot4(h, h);
    }
    L::head_reduce(d);
    if (ok && q == 0 && nu) nu[row] = fmaxf(sqrtf(d[0]), eps);
  }
}

// ---------------------------------------------------------------- backward


template <int K, int MODEL>
__device__ __forceinline__ void bwd_store(const AvBwd& A, int64_t row, int64_t grow, int q,
                                          const float4 (&dh)[RowLayout<K, 1>::VPL],
                                          const float4 (&acc)[RowLayout<K, 1>::VPL], bool write) {
  using L = RowLayout<K, 1>;
  if (MODEL == VA) {
    if (write) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) st4(A.dH + row * K + L::col(v, q), dh[v]);
    }
    return;
  }
  // AGNN: dH_j = acc_j + (dH^_j - (dH^_j . H^_j) H^_j) / nu_j  (nu const on the eps branch)
  const float nuj = A.rec[grow].x;
  float4 Hj[L::VPL];
  float pr[L::VPL];
#pragma unroll
  for (int v = 0; v < L::VPL; ++v) {
    // (BF16 mode, heavy-row merge: the rounded row H~_j the layer computes on)
    Hj[v] = A.H16 ? ldg4(A.H16 + grow * K + L::col(v, q)) : ldg4(A.H + grow * K + L::col(v, q));
    pr[v] = dot4(dh[v], Hj[v]);
  }
  L::head_reduce(pr);  // every lane participates (uniform)
  const bool on_eps = !(nuj > A.eps);
  const float inv = 1.f / nuj;
  const float proj = on_eps ? 0.f : pr[0] * inv * inv;  // (dH^.H^) / nu_j  applied to H_j
  if (write) {
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      float4 gv = fma4(-proj, Hj[v], dh[v]);
      gv = fma4(inv, gv, acc[v]);
      st4(A.dH + row * K + L::col(v, q), gv);
    }
  }
}

// ROLE: 0 = both roles over the symmetric CSR; 1 = row role only over the CSR of a
// directed pattern (partial -> A.dhp); 2 = column role only over its CSC (items are
// columns j, it.col the rows i with stored (i,j)), adding A.dhp before the epilogue
template <int K, int MODEL, int U, int ROLE = 0>
__global__ void __launch_bounds__(kSparseThreads) av_bwd_kernel(Items it, AvBwd A) {
  constexpr bool RR = ROLE != 2, CR = ROLE != 1;
  using L = RowLayout<K, 1>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const float beta = A.beta;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_range<K>(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float4 Hj[L::VPL], Mj[L::VPL], dh[L::VPL], acc[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) {
      Hj[v] = ldg4(A.H + grow * K + L::col(v, q));
      Mj[v] = ldg4(A.M + grow * K + L::col(v, q));
      dh[v] = acc[v] = f4(0.f);
    }
    const float4 rj = (MODEL == AG) ? __ldg(A.rec + grow) : f4(0.f);
    const float sj = (MODEL == AG) ? beta / rj.x : 0.f;
    for (int64_t e0 = beg; e0 < end; e0 += 32) {
      const int cnt = (int)(end - e0 < 32 ? end - e0 : 32);
      const int myc = lane < cnt ? __ldg(it.col + e0 + lane) : 0;
      for (int b = 0; b < cnt; b += L::GROUPS * U) {
        float4 Hi[U][L::VPL], Mi[U][L::VPL], ri[U];
        bool val[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int se = b + u * L::GROUPS + g;
          val[u] = se < cnt;
          const int64_t i = __shfl_sync(FULL, myc, se & 31);
#pragma unroll
          for (int v = 0; v < L::VPL; ++v) {
            Hi[u][v] = val[u] ? ldg4(A.H + i * K + L::col(v, q)) : f4(0.f);
            Mi[u][v] = (CR && val[u]) ? ldg4(A.M + i * K + L::col(v, q)) : f4(0.f);
          }
          ri[u] = (MODEL == AG && val[u]) ? __ldg(A.rec + i) : f4(1.f);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          float s[L::VPL], d1[L::VPL], d2[L::VPL];
#pragma unroll
          for (int v = 0; v < L::VPL; ++v) {
            s[v] = dot4(Hj[v], Hi[u][v]);    // H_j . H_i
            d1[v] = dot4(Mj[v], Hi[u][v]);   // M_j . H_i  (row role)
            d2[v] = dot4(Mi[u][v], Hj[v]);   // M_i . H_j  (column role)
          }
          if (MODEL == AG || CR) L::head_reduce(s);
          if (RR) L::head_reduce(d1);
          if (CR) L::head_reduce(d2);
          if (!val[u]) continue;
          if (MODEL == VA) {
            const float c1 = (RR ? d1[0] : 0.f) + (CR ? d2[0] : 0.f);
#pragma unroll
            for (int v = 0; v < L::VPL; ++v) {
              dh[v] = fma4(c1, Hi[u][v], dh[v]);
              if (CR) dh[v] = fma4(s[0], Mi[u][v], dh[v]);
            }
          } else {
            const float inv_nui = 1.f / ri[u].x;
            const float c = sj * s[0] * inv_nui;                        // beta cos(H_j, H_i)
            float dc = 0.f, aij = 0.f;
            if (RR) {
              const float aji = ex2((c - rj.y) * kLog2e) * rj.z;        // alpha_ji (row j)
              dc = aji * (d1[0] - rj.w);
            }
            if (CR) {
              aij = ex2((c - ri[u].y) * kLog2e) * ri[u].z;              // alpha_ij (row i)
              dc += aij * (d2[0] - ri[u].w);
            }
            dc *= beta;
#pragma unroll
            for (int v = 0; v < L::VPL; ++v) {
              dh[v] = fma4(dc * inv_nui, Hi[u][v], dh[v]);   // dH^_j += dc H^_i
              if (CR) acc[v] = fma4(aij, Mi[u][v], acc[v]);
            }
          }
        }
      }
    }
#pragma unroll
    for (int off = L::LANES; off < 32; off <<= 1) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        dh[v].x += __shfl_xor_sync(FULL, dh[v].x, off);
        dh[v].y += __shfl_xor_sync(FULL, dh[v].y, off);
        dh[v].z += __shfl_xor_sync(FULL, dh[v].z, off);
        dh[v].w += __shfl_xor_sync(FULL, dh[v].w, off);
        if (MODEL == AG && CR) {
          acc[v].x += __shfl_xor_sync(FULL, acc[v].x, off);
          acc[v].y += __shfl_xor_sync(FULL, acc[v].y, off);
          acc[v].z += __shfl_xor_sync(FULL, acc[v].z, off);
          acc[v].w += __shfl_xor_sync(FULL, acc[v].w, off);
        }
      }
    }
    if (slot >= 0) {
      if (g == 0) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) {
          st4(A.pacc + slot * 2 * K + L::col(v, q), dh[v]);
          if (MODEL == AG && CR) st4(A.pacc + slot * 2 * K + K + L::col(v, q), acc[v]);
        }
      }
    } else if (ROLE == 1) {
      if (g == 0) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) st4(A.dhp + row * K + L::col(v, q), dh[v]);
      }
    } else {
      if (ROLE == 2) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) dh[v] = add4(ldg4(A.dhp + row * K + L::col(v, q)), dh[v]);
      }
      bwd_store<K, MODEL>(A, row, grow, q, dh, acc, g == 0);
    }
  }
}

template <int K, int MODEL, int ROLE = 0>
__global__ void __launch_bounds__(kSparseThreads) av_bwd_merge_kernel(Items it, AvBwd A) {
  using L = RowLayout<K, 1>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t h = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; h < it.n_heavy; h += nw) {
    const int64_t row = it.heavy_rows[h], grow = it.row_begin + row;
    float4 dh[L::VPL], acc[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v) dh[v] = acc[v] = f4(0.f);
    for (int64_t s = it.heavy_off[h]; s < it.heavy_off[h + 1]; ++s) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) {
        dh[v] = add4(dh[v], ldg4(A.pacc + s * 2 * K + L::col(v, q)));
        if (MODEL == AG && ROLE != 1) acc[v] = add4(acc[v], ldg4(A.pacc + s * 2 * K + K + L::col(v, q)));
      }
    }
    if (ROLE == 1) {
      if (g == 0) {
#pragma unroll
        for (int v = 0; v < L::VPL; ++v) st4(A.dhp + row * K + L::col(v, q), dh[v]);
      }
      continue;
    }
    if (ROLE == 2) {
#pragma unroll
      for (int v = 0; v < L::VPL; ++v) dh[v] = add4(ldg4(A.dhp + row * K + L::col(v, q)), dh[v]);
    }
    bwd_store<K, MODEL>(A, row, grow, q, dh, acc, g == 0);
  }
}

// G = dH_out (.) sigma'(Z)   (elementwise, n_local x k_out)
__global__ void grad_act_kernel(const float* __restrict__ dHout, const float* __restrict__ Z,
                                int64_t count4, int act, float* __restrict__ G) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count4;
       i += (int64_t)gridDim.x * blockDim.x) {
    const float4 z = ldg4(Z + 4 * i), d = ldg4(dHout + 4 * i);
    st4(G + 4 * i, make_float4(d.x * act_grad(act, z.x), d.y * act_grad(act, z.y),
                               d.z * act_grad(act, z.z), d.w * act_grad(act, z.w)));
  }
}

// rec_i = {nu_i, |beta|, 1/l_i, delta_i = M_i . X_i}   (AGNN; TM = bf16: M~, reading B2)
template <int K, typename TM = float>
__global__ void __launch_bounds__(kSparseThreads)
agnn_rec_kernel(int64_t n_local, int64_t row_begin, const TM* __restrict__ M,
                const float* __restrict__ X, const float* __restrict__ nu,
                const float* __restrict__ l, float bound, float4* __restrict__ rec) {
  using L = RowLayout<K, 1>;
  const int lane = threadIdx.x & 31, g = lane / L::LANES, q = lane % L::LANES;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t slots = (n_local + L::GROUPS - 1) / L::GROUPS;
  for (int64_t rs = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; rs < slots; rs += nw) {
    const int64_t row = rs * L::GROUPS + g;
    const bool ok = row < n_local;
    const int64_t grow = row_begin + row;
    float d[L::VPL];
#pragma unroll
    for (int v = 0; v < L::VPL; ++v)
      d[v] = ok ? dot4(ldg4(M + grow * K + L::col(v, q)), ldg4(X + row * K + L::col(v, q))) : 0.f;
    L::head_reduce(d);
    if (ok && q == 0) {
      const float lv = l[row];
      rec[grow] = make_float4(nu[grow], bound, lv > 0.f ? 1.f / lv : 0.f, d[0]);
    }
  }
}

__global__ void av_debug_kernel(const int64_t* __restrict__ rp, int64_t n_local,
                                const int32_t* __restrict__ col, int64_t row_begin,
                                const float* __restrict__ H, const bf16* __restrict__ H16, int K,
                                const float* __restrict__ nu,
                                const float* __restrict__ l, int model, float beta, float bound,
                                const int64_t* __restrict__ pos, int64_t count,
                                float* __restrict__ out) {
  const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= count) return;
  const int64_t e = pos[t];
  int64_t lo = 0, hi = n_local;
  while (hi - lo > 1) {
    const int64_t mid = (lo + hi) / 2;
    if (rp[mid] <= e) lo = mid; else hi = mid;
  }
  const int64_t i = row_begin + lo, j = col[e];
  float s = 0.f;
  if (H16)
    for (int c = 0; c < K; ++c)
      s = fmaf(__bfloat162float(H16[i * K + c]), __bfloat162float(H16[j * K + c]), s);
  else
    for (int c = 0; c < K; ++c) s = fmaf(H[i * K + c], H[j * K + c], s);
  if (model == VA) {
    out[t] = s;
  } else {
    out[t] = expf(beta * s / (nu[i] * nu[j]) - bound) / l[lo];
  }
}

bool av_bf16(const agnn_layer_desc& d) { return d.prec == AGNN_PREC_BF16; }

struct SavedAv {
  float *Hfull, *nu, *X, *Z, *l;
  bf16* H16;  // BF16 mode (reading B2): H~ [n x k_in] (replicated), replaces Hfull
};
SavedAv carve_saved(const Plan& p, const agnn_layer_desc& d, void* base, size_t* total) {
  Carver c(base);
  SavedAv s;
  s.H16 = c.take<bf16>(av_bf16(d) ? (size_t)p.n * d.k_in : 0);
  s.Hfull = c.take<float>(p.world > 1 && !av_bf16(d) ? (size_t)p.n * d.k_in : 0);
  s.nu = c.take<float>(d.kind == AGNN_AGNN ? (size_t)p.n : 0);
  s.X = c.take<float>((size_t)p.n_local * d.k_in);
  s.Z = c.take<float>((size_t)p.n_local * d.k_out);
  s.l = c.take<float>(d.kind == AGNN_AGNN ? (size_t)p.n_local : 0);
  if (total) *total = c.off + 256;
  return s;
}

struct WsAv {
  float *pacc, *pl, *G, *M, *gemm, *WT, *dhp;
  float4* rec;
  int* hcnt;  // SpMMM: completed chunks per heavy row
  void* saved_inf;
  bf16* M16;  // BF16 mode (reading B2): M~ [n x k_in] (replicated), replaces M
};
WsAv carve_ws(const Plan& p, const agnn_layer_desc& d, void* base, size_t* total) {
  Carver c(base);
  WsAv w;
  size_t sv = 0;
  carve_saved(p, d, nullptr, &sv);
  // replicated (n-row) arrays first (same offsets on every rank; peer exchange)
  w.M16 = c.take<bf16>(av_bf16(d) ? (size_t)p.n * d.k_in : 0);
  // (BF16 mode: fp32 scratch of the local rows, used only by shapes without tcgen05)
  w.M = c.take<float>(av_bf16(d) ? (size_t)p.n_local * d.k_in : (size_t)p.n * d.k_in);
  w.rec = c.take<float4>(d.kind == AGNN_AGNN ? (size_t)p.n : 0);
  w.saved_inf = c.take<char>(sv);  // its replicated prefix (H_full, nu) too
  w.pacc = c.take<float>((size_t)p.max_chunks() * 2 * d.k_in);
  w.pl = c.take<float>((size_t)p.max_chunks());
  w.dhp = c.take<float>(p.csc_ptr ? (size_t)p.n_local * d.k_in : 0);
  w.G = c.take<float>((size_t)p.n_local * d.k_out);
  w.gemm = c.take<float>(gemm_tn_ws_floats(d.k_in, d.k_out));
  w.WT = c.take<float>((size_t)d.k_in * d.k_out);
  w.hcnt = c.take<int>(p.spmmm ? (size_t)p.n_heavy : 0);
  if (total) *total = c.off + 256;
  return w;
}

}  // namespace

agnn_status av_saved_bytes(const Plan& p, const agnn_layer_desc& d, size_t* b) {
  carve_saved(p, d, nullptr, b);
  return AGNN_OK;
}
agnn_status av_workspace_bytes(const Plan& p, const agnn_layer_desc& d, size_t* b) {
  carve_ws(p, d, nullptr, b);
  return AGNN_OK;
}

#define AGNN_AV_DISPATCH(K_, CALL)                                           \
  do {                                                                       \
    if (K_ == 16) { constexpr int K = 16; CALL; }                           \
    else if (K_ == 32) { constexpr int K = 32; CALL; }                      \
    else if (K_ == 64) { constexpr int K = 64; CALL; }                      \
    else if (K_ == 128) { constexpr int K = 128; CALL; }                    \
    else if (K_ == 256) { constexpr int K = 256; CALL; }                    \
    else return fail(AGNN_EUNSUPPORTED, "AGNN/VA: k_in must be 16/32/64/128/256"); \
  } while (0)

template <int K>
constexpr int av_fwd_unroll() { return K >= 256 ? 2 : 4; }
template <int K>
constexpr int av_bwd_unroll() { return K >= 256 ? 1 : 2; }

agnn_status av_forward(const Plan& p, const agnn_layer_desc& d, const float* W, const float* H_in,
                       float* H_out, void* saved, void* ws, cudaStream_t s) {
  WsAv w = carve_ws(p, d, ws, nullptr);
  SavedAv sv = carve_saved(p, d, saved ? saved : w.saved_inf, nullptr);
  const int K_ = d.k_in;
  const bool ag = d.kind == AGNN_AGNN;
  agnn_status st;
  const float* Hf = H_in;
  const bool b16 = av_bf16(d);
  if (b16) {
    if (p.directed() || !(K_ == 128 || K_ == 256))
      return fail(AGNN_EUNSUPPORTED, "AGNN/VA BF16: symmetric patterns with k_in = 128 / 256");
    AGNN_AV_DISPATCH(K_, (av_round_kernel<K><<<grid_of(av_round_kernel<K>), kSparseThreads, 0, s>>>(
                             H_in, p.n_local, d.eps, sv.H16 + p.row_begin * d.k_in,
                             ag ? sv.nu + p.row_begin : nullptr)));
    AGNN_LAUNCH_CHECK("av_round_kernel");
    if (p.world > 1) {
      const RowArray ra[2] = {{reinterpret_cast<float*>(sv.H16), d.k_in / 2}, {sv.nu, 1}};
      if ((st = allgather_rows(p, ra, ag ? 2 : 1, s)) != AGNN_OK) return st;
    }
  } else if (ag) {
    AGNN_AV_DISPATCH(K_, (nu_kernel<K><<<grid_of(nu_kernel<K>), kSparseThreads, 0, s>>>(
                             H_in, p.n_local, d.eps, sv.nu + p.row_begin)));
    AGNN_LAUNCH_CHECK("nu_kernel");
  }
  if (p.world > 1 && !b16) {
    AGNN_CUDA_TRY(cudaMemcpyAsync(sv.Hfull + p.row_begin * d.k_in, H_in,
                                  sizeof(float) * p.n_local * d.k_in, cudaMemcpyDeviceToDevice, s));
    const RowArray ra[2] = {{sv.Hfull, d.k_in}, {sv.nu, 1}};
    if ((st = allgather_rows(p, ra, ag ? 2 : 1, s)) != AGNN_OK) return st;
    Hf = sv.Hfull;
  }
  Items it = items_of(p);
  AvFwd A{Hf, b16 ? sv.H16 : nullptr, sv.nu, d.beta, fabsf(d.beta), sv.X, sv.l, w.pacc, w.pl};
  if (p.spmmm && K_ == 128 && d.k_out == 128) {
    // SpMMM (S8(f) f2): aggregation (heavy-row chunks and their merge included) and
    // the projection by W in one kernel, X staying on chip
    const Items ith = l2_hinted(it, p, (b16 ? 2 : 4) * (int64_t)K_ + (ag ? 4 : 0));
    return av_fwd_spmmm(ith, ag, A, W, saved ? sv.Z : nullptr, H_out, w.hcnt, (int)d.act,
                        saved != nullptr, s);
  }
  if (K_ == 128 || K_ == 256) {
    // gathered per entry: an H_j row (+ nu_j)
    const Items ith = l2_hinted(it, p, (b16 ? 2 : 4) * (int64_t)K_ + (ag ? 4 : 0));
    if ((st = av_fwd_batched(ith, K_, ag, A, s)) != AGNN_OK) return st;
  } else if (it.n_chunks + it.n_light > 0) {
    if (ag) AGNN_AV_DISPATCH(K_, (av_fwd_kernel<K, AG, av_fwd_unroll<K>()>
                                  <<<grid_of(av_fwd_kernel<K, AG, av_fwd_unroll<K>()>),
                                     kSparseThreads, 0, s>>>(it, A)));
    else AGNN_AV_DISPATCH(K_, (av_fwd_kernel<K, VA, av_fwd_unroll<K>()>
                               <<<grid_of(av_fwd_kernel<K, VA, av_fwd_unroll<K>()>),
                                  kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("av_fwd_kernel");
  }
  if (it.n_heavy > 0) {
    if (ag) AGNN_AV_DISPATCH(K_, (av_fwd_merge_kernel<K, AG>
                                  <<<kNumSMs * 2, kSparseThreads, 0, s>>>(it, A)));
    else AGNN_AV_DISPATCH(K_, (av_fwd_merge_kernel<K, VA>
                               <<<kNumSMs * 2, kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("av_fwd_merge_kernel");
  }
  // Z = X W ; H_out = sigma(Z)   (B = W^T as [k_out x k_in] for the tensor-core path)
  if ((st = transpose(W, d.k_in, d.k_out, w.WT, s)) != AGNN_OK) return st;
  return gemm_rows(sv.X, p.n_local, d.k_in, w.WT, true, d.k_out, saved ? sv.Z : nullptr, d.k_out,
                   nullptr, s, H_out, (int)d.act);
}

agnn_status av_backward(const Plan& p, const agnn_layer_desc& d, const float* W,
                        const float* H_in, const void* saved, const float* dH_out, float* dH_in,
                        float* dW, void* ws, cudaStream_t s) {
  const bool directed = p.directed();
  if (directed && !p.csc_ptr)
    return fail(AGNN_EUNSUPPORTED,
                "agnn_backward: a directed pattern needs world == 1 and every row in the plan");
  WsAv w = carve_ws(p, d, ws, nullptr);
  SavedAv sv = carve_saved(p, d, const_cast<void*>(saved), nullptr);
  const int K_ = d.k_in;
  const bool ag = d.kind == AGNN_AGNN;
  agnn_status st;
  const int64_t c4 = p.n_local * d.k_out / 4;
  if (c4 > 0) {
    grad_act_kernel<<<kNumSMs * 8, kSparseThreads, 0, s>>>(dH_out, sv.Z, c4, (int)d.act, w.G);
    AGNN_LAUNCH_CHECK("grad_act_kernel");
  }
  // Y = dW = X^T G  (= H^T (A^T (.) H_x) G for VA, Eq. 13)
  if ((st = gemm_tn(sv.X, p.n_local, d.k_in, w.G, d.k_out, dW, w.gemm, s)) != AGNN_OK) return st;
  if (p.world > 1 && (st = allreduce_sum(p, dW, (int64_t)d.k_in * d.k_out, s)) != AGNN_OK) return st;
  if (!dH_in) return AGNN_OK;
  // M = G W^T (Eq. 12) for the local rows; with P > 1 the rows the other ranks
  // reference (and AGNN's records) then go to their replicas (comm.cu).  BF16 mode
  // (reading B2): the GEMM epilogue stores M~ = bf16(M), used everywhere after.
  const bool b16 = av_bf16(d);
  if (b16) {
    if ((st = gemm_rows_bf16(w.G, p.n_local, d.k_out, W, d.k_in, w.M16 + p.row_begin * d.k_in,
                             d.k_in, nullptr, w.M, s)) != AGNN_OK)
      return st;
    if (ag) {
      AGNN_AV_DISPATCH(K_, (agnn_rec_kernel<K, bf16><<<grid_of(agnn_rec_kernel<K, bf16>),
                                                      kSparseThreads, 0, s>>>(
                               p.n_local, p.row_begin, w.M16, sv.X, sv.nu, sv.l, fabsf(d.beta),
                               w.rec)));
      AGNN_LAUNCH_CHECK("agnn_rec_kernel");
    }
    if (p.world > 1) {
      const RowArray ra[2] = {{reinterpret_cast<float*>(w.M16), d.k_in / 2},
                              {reinterpret_cast<float*>(w.rec), 4}};
      if ((st = allgather_rows(p, ra, ag ? 2 : 1, s)) != AGNN_OK) return st;
    }
  } else {
    float* Mloc = w.M + p.row_begin * d.k_in;
    if ((st = gemm_rows(w.G, p.n_local, d.k_out, W, true, d.k_in, Mloc, d.k_in, nullptr, s)) !=
        AGNN_OK)
      return st;
    if (ag) {
      AGNN_AV_DISPATCH(K_, (agnn_rec_kernel<K><<<grid_of(agnn_rec_kernel<K>), kSparseThreads, 0, s>>>(
                               p.n_local, p.row_begin, w.M, sv.X, sv.nu, sv.l, fabsf(d.beta), w.rec)));
      AGNN_LAUNCH_CHECK("agnn_rec_kernel");
    }
    if (p.world > 1) {
      const RowArray ra[2] = {{w.M, d.k_in}, {reinterpret_cast<float*>(w.rec), 4}};
      if ((st = allgather_rows(p, ra, ag ? 2 : 1, s)) != AGNN_OK) return st;
    }
  }
  const float* Hf = p.world > 1 ? sv.Hfull : H_in;
  Items it = items_of(p);
  AvBwd A{Hf, w.M, b16 ? sv.H16 : nullptr, b16 ? w.M16 : nullptr, w.rec, d.beta, d.eps, dH_in,
          w.pacc, w.dhp};
  if (directed) {
#define AV_PASS(ROLE_, ITEMS)                                                                      \
    do {                                                                                           \
      const Items itr = (ITEMS);                                                                   \
      if (itr.n_chunks + itr.n_light > 0) {                                                        \
        if (ag) AGNN_AV_DISPATCH(K_, (av_bwd_kernel<K, AG, av_bwd_unroll<K>(), ROLE_>               \
                                      <<<grid_of(av_bwd_kernel<K, AG, av_bwd_unroll<K>(), ROLE_>),   \
                                         kSparseThreads, 0, s>>>(itr, A)));                        \
        else AGNN_AV_DISPATCH(K_, (av_bwd_kernel<K, VA, av_bwd_unroll<K>(), ROLE_>                  \
                                   <<<grid_of(av_bwd_kernel<K, VA, av_bwd_unroll<K>(), ROLE_>),      \
                                      kSparseThreads, 0, s>>>(itr, A)));                           \
        AGNN_LAUNCH_CHECK("av_bwd_kernel");                                                        \
      }                                                                                            \
      if (itr.n_heavy > 0) {                                                                       \
        if (ag) AGNN_AV_DISPATCH(K_, (av_bwd_merge_kernel<K, AG, ROLE_>                             \
                                      <<<kNumSMs * 2, kSparseThreads, 0, s>>>(itr, A)));           \
        else AGNN_AV_DISPATCH(K_, (av_bwd_merge_kernel<K, VA, ROLE_>                                \
                                   <<<kNumSMs * 2, kSparseThreads, 0, s>>>(itr, A)));              \
        AGNN_LAUNCH_CHECK("av_bwd_merge_kernel");                                                  \
      }                                                                                            \
    } while (0)
    AV_PASS(1, it);                  // row role over the CSR  -> dhp
    AV_PASS(2, items_of_csc(p));     // column role over the CSC (+ dhp) -> dH
#undef AV_PASS
    return AGNN_OK;
  }
  if (K_ == 128 || K_ == 256) {
    // gathered per entry: the H_i and M_i rows (+ the record)
    const Items ith = l2_hinted(it, p, (b16 ? 4 : 8) * (int64_t)K_ + (ag ? 16 : 0));
    if ((st = av_bwd_batched(ith, K_, ag, A, s)) != AGNN_OK) return st;
  } else if (it.n_chunks + it.n_light > 0) {
    if (ag) AGNN_AV_DISPATCH(K_, (av_bwd_kernel<K, AG, av_bwd_unroll<K>()>
                                  <<<grid_of(av_bwd_kernel<K, AG, av_bwd_unroll<K>()>),
                                     kSparseThreads, 0, s>>>(it, A)));
    else AGNN_AV_DISPATCH(K_, (av_bwd_kernel<K, VA, av_bwd_unroll<K>()>
                               <<<grid_of(av_bwd_kernel<K, VA, av_bwd_unroll<K>()>),
                                  kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("av_bwd_kernel");
  }
  if (it.n_heavy > 0) {
    if (ag) AGNN_AV_DISPATCH(K_, (av_bwd_merge_kernel<K, AG>
                                  <<<kNumSMs * 2, kSparseThreads, 0, s>>>(it, A)));
    else AGNN_AV_DISPATCH(K_, (av_bwd_merge_kernel<K, VA>
                               <<<kNumSMs * 2, kSparseThreads, 0, s>>>(it, A)));
    AGNN_LAUNCH_CHECK("av_bwd_merge_kernel");
  }
  return AGNN_OK;
}

agnn_status av_debug_attention(const Plan& p, const agnn_layer_desc& d, const void* saved,
                               const float* H_in, const int64_t* pos, int64_t count, float* out,
                               cudaStream_t s) {
  if (!saved) return fail(AGNN_EINVAL, "debug_attention: saved == NULL");
  if (count <= 0) return AGNN_OK;
  SavedAv sv = carve_saved(p, d, const_cast<void*>(saved), nullptr);
  const float* Hf = p.world > 1 ? sv.Hfull : H_in;
  const bf16* H16 = av_bf16(d) ? sv.H16 : nullptr;
  if (!Hf && !H16) return fail(AGNN_EINVAL, "debug_attention: AGNN/VA need H_in on one GPU");
  av_debug_kernel<<<(unsigned)((count + 255) / 256), 256, 0, s>>>(
      p.row_ptr, p.n_local, p.col_idx, p.row_begin, Hf, H16, d.k_in, sv.nu, sv.l,
      d.kind == AGNN_AGNN ? AG : VA, d.beta, fabsf(d.beta), pos, count, out);
  AGNN_LAUNCH_CHECK("av_debug_kernel");
  return AGNN_OK;
}

}  // namespace agnn
