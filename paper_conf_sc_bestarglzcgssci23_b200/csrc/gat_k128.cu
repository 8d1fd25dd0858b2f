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
// Backward, per row j, edges in batches of B (<= lanes per head):
//   warp-parallel: gather P_i, G_i slices; partial dots G_j.P_i and G_i.P_j;
//   a transposed butterfly reduction leaves each lane with both full dots of
//   ONE edge of its head; lane-parallel scalar work (the two alpha recomputes,
//   dc_ji, dc_ij); alpha_ij is broadcast back for acc_j += alpha_ij G_i.
#include "gat_args.cuh"

namespace agnn {
namespace {

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

__device__ __forceinline__ void item_of(const Items& it, int64_t w, int64_t& row, int64_t& beg,
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

// ---------------------------------------------------------------- forward
template <int NH, int U>
__global__ void __launch_bounds__(256)
gat_fwd_k128_kernel(Items it, const float* __restrict__ P, const float* __restrict__ st,
                    float slope, int act, GatFwdOut o) {
  constexpr int D = K / NH, HL = D / 4;
  __shared__ float sPw[8][NH][33];  // +1: heads read different rows without bank conflicts
  __shared__ int sJ[8][32];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int hv = lane / HL, cq = lane * 4;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    float si[NH], mr[NH], lp[NH];
    load_n<NH>(st + grow * (2 * NH), si);
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      mr[h] = -INFINITY;
      lp[h] = 0.f;
    }
    float4 acc = f4(0.f);
    for (int64_t b0 = beg; b0 < end; b0 += 32) {
      const int cnt = (int)(end - b0 < 32 ? end - b0 : 32);
      const bool valid = lane < cnt;
      const int j = valid ? __ldg(it.col + b0 + lane) : 0;
      float tj[NH];
      load_n<NH>(st + (int64_t)j * (2 * NH) + NH, tj);
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
        lp[h] *= sc;
        if (h == hv) sch = sc;
        mr[h] = mn;
        const float p = valid ? ex2(e - mn) : 0.f;
        lp[h] += p;
        sPw[wib][h][lane] = p;
      }
      acc = mul4(sch, acc);
      sJ[wib][lane] = j;
      __syncwarp();
      for (int k = 0; k < cnt; k += U) {
        float4 pv[U];
        float pw[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int kk = k + u;
          if (kk < cnt) {
            pv[u] = ldg4(P + (int64_t)sJ[wib][kk] * K + cq);
            pw[u] = sPw[wib][hv][kk];
          } else {
            pv[u] = f4(0.f);
            pw[u] = 0.f;
          }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) acc = fma4(pw[u], pv[u], acc);
      }
      __syncwarp();
    }
    float l[NH];
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      float x = lp[h];
#pragma unroll
      for (int off = 16; off > 0; off >>= 1) x += __shfl_xor_sync(FULL, x, off);
      l[h] = x;
    }
    float lh = l[0], mh = mr[0];
#pragma unroll
    for (int h = 1; h < NH; ++h)
      if (h == hv) {
        lh = l[h];
        mh = mr[h];
      }
    if (slot >= 0) {
      st4(o.pacc + slot * K + cq, acc);
      if (lane == 0) {
#pragma unroll
        for (int h = 0; h < NH; ++h) {
          o.pm[slot * NH + h] = mr[h];
          o.pl[slot * NH + h] = l[h];
        }
      }
    } else {
      const float4 z = mul4(lh > 0.f ? 1.f / lh : 0.f, acc);
      if (o.Z) st4(o.Z + row * K + cq, z);
      st4(o.Hout + row * K + cq, act_fwd4(act, z));
      if (o.m && lane == 0) {
#pragma unroll
        for (int h = 0; h < NH; ++h) {
          o.m[row * NH + h] = l[h] > 0.f ? mr[h] : 0.f;
          o.l[row * NH + h] = l[h];
        }
      }
      (void)mh;
    }
  }
}

// ---------------------------------------------------------------- backward
template <int B>
struct Transpose {
  static constexpr int T = (B >= 8) ? 3 : (B >= 4) ? 2 : (B >= 2) ? 1 : 0;
  // edge index held by lane-in-group ql after the transposed reduction
  __device__ static __forceinline__ int edge_of(int ql) {
    int b = 0;
#pragma unroll
    for (int s = 0; s < T; ++s) b |= ((ql >> s) & 1) * (B >> (s + 1));
    return b;
  }
  // lane-in-group that holds edge b
  __device__ static __forceinline__ int lane_of(int b) {
    int q = 0;
#pragma unroll
    for (int s = 0; s < T; ++s) q |= ((b / (B >> (s + 1))) & 1) << s;
    return q;
  }
  // x[0..B) partial sums over the HL lanes of a head group -> x[0] = full sum of
  // element edge_of(lane % HL), every lane
  template <int HL>
  __device__ static __forceinline__ void reduce(float (&x)[B], int lane) {
    int len = B;
#pragma unroll
    for (int s = 0; s < T; ++s) {
      const int o = 1 << s;
      const bool upper = (lane & o) != 0;
      len >>= 1;
#pragma unroll
      for (int k = 0; k < B / 2; ++k) {
        if (k < len) {
          const float keep = upper ? x[k + len] : x[k];
          const float send = upper ? x[k] : x[k + len];
          x[k] = keep + __shfl_xor_sync(FULL, send, o);
        }
      }
    }
#pragma unroll
    for (int o = B; o < HL; o <<= 1) x[0] += __shfl_xor_sync(FULL, x[0], o);
  }
};

template <int NH, int B>
__global__ void __launch_bounds__(256, 3)
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
  float4 da1 = f4(0.f), da2 = f4(0.f);

  for (int64_t w = gw; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    const float4 Pj = ldg4(A.P + grow * K + cq);
    const float4 Gj = ldg4(A.G + grow * K + cq);
    const float4 rj = __ldg(A.rec + grow * NH + hv);        // {s_j, m_j, 1/l_j, delta_j}
    const float tj = __ldg(A.st + grow * (2 * NH) + NH + hv);
    float4 acc = f4(0.f);
    float dsp = 0.f, dtp = 0.f;
    int cidx = 0;
    for (int64_t b0 = beg; b0 < end; b0 += B) {
      const int off32 = (int)((b0 - beg) & 31);
      if (off32 == 0) {
        const int64_t e = b0 + lane;
        cidx = e < end ? __ldg(it.col + e) : 0;
      }
      const int cnt = (int)(end - b0 < B ? end - b0 : B);
      float4 Pi[B], Gi[B];
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const int64_t i = __shfl_sync(FULL, cidx, off32 + b);
        if (b < cnt) {
          Pi[b] = ldg4(A.P + i * K + cq);
          Gi[b] = ldg4(A.G + i * K + cq);
        } else {
          Pi[b] = Gi[b] = f4(0.f);
        }
      }
      // scalar operands of the edge this lane will own after the reduction
      const int64_t im = __shfl_sync(FULL, cidx, off32 + my_b);
      const bool vm = my_b < cnt;
      const float4 ri = vm ? __ldg(A.rec + im * NH + hv) : f4(0.f);
      const float ti = vm ? __ldg(A.st + im * (2 * NH) + NH + hv) : 0.f;
      float x1[B], x2[B];
#pragma unroll
      for (int b = 0; b < B; ++b) {
        x1[b] = dot4(Gj, Pi[b]);  // G_j . P_i  (row role)
        x2[b] = dot4(Gi[b], Pj);  // G_i . P_j  (column role)
      }
      TR::template reduce<HL>(x1, lane);
      TR::template reduce<HL>(x2, lane);
      // row role: entry (j,i) of row j
      const float pre = rj.x + ti;
      const float e = fmaxf(pre, slope * pre);
      const float aji = ex2(e - rj.y) * rj.z;
      const float dcji = aji * (pre > 0.f ? 1.f : slope) * (x1[0] - rj.w);
      // column role: entry (i,j) of row i
      const float pre2 = ri.x + tj;
      const float e2 = fmaxf(pre2, slope * pre2);
      float aij = ex2(e2 - ri.y) * ri.z;
      const float dcij = aij * (pre2 > 0.f ? 1.f : slope) * (x2[0] - ri.w);
      if (vm && owner) {
        dsp += dcji;
        dtp += dcij;
      }
      if (!vm) aij = 0.f;
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const float ab = __shfl_sync(FULL, aij, gbase + TR::lane_of(b));
        acc = fma4(ab, Gi[b], acc);
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

agnn_status gat_fwd_k128(const Items& it, int heads, const float* P, const float* st, float slope,
                         int act, const GatFwdOut& o, cudaStream_t s) {
  if (it.n_chunks + it.n_light == 0) return AGNN_OK;
  AGNN_K128_DISPATCH(heads, ({
    gat_fwd_k128_kernel<NH, 8><<<grid_for(gat_fwd_k128_kernel<NH, 8>), 256, 0, s>>>(
        it, P, st, slope, act, o);
    AGNN_LAUNCH_CHECK("gat_fwd_kernel");
  }));
  return AGNN_OK;
}

agnn_status gat_bwd_k128(const Items& it, int heads, const GatBwdArgs& A, int64_t* warps,
                         cudaStream_t s) {
  *warps = 0;
  AGNN_K128_DISPATCH(heads, ({
    constexpr int B = bwd_batch<NH>();
    const int grid = grid_for(gat_bwd_k128_kernel<NH, B>);
    gat_bwd_k128_kernel<NH, B><<<grid, 256, 0, s>>>(it, A);
    AGNN_LAUNCH_CHECK("gat_bwd_kernel");
    *warps = (int64_t)grid * 8;
  }));
  return AGNN_OK;
}

}  // namespace agnn
