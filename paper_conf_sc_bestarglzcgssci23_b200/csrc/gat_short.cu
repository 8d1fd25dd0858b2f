// gat_short.cu — GAT k' = 128 sparse kernels for SHORT rows (degree <= the plan's
// short_max, default 32).  Same arithmetic as gat_k128.cu (PAPER.md:177 forward
// with the graph softmax of :191; :250-254 backward with Psi^T, readings A11/A12;
// scores in log2 units), different work decomposition.
//
// Why: half the rows of a Kronecker graph have degree < 4 (median
// 2-3) and hold ~2 % of the edges, but a warp-per-row kernel pays a chain of
// dependent loads per row (row id -> row_ptr -> column ids -> gathered rows)
// for a handful of edges: measured on C5 (bf16), rows of degree < 64 were 12 % of
// the edges and ~27 % of the sparse-kernel time.  Here a warp carries 32/SUB
// rows at once — SUB lanes per row, 128/SUB columns per lane (16-byte loads) —
// so the latency chains of 4 rows overlap, and every lane computes the scalar
// work of its own head redundantly (no cross-lane softmax reductions at all).
//
// Forward, per row i: edges in batches of U; per batch one max / rescale of the
//   running (m, l, acc) (online softmax, as gat_k128.cu per 32-edge batch).
// Backward, per row j: per edge both roles of the stored entry (j,i) (symmetric
//   pattern): dot products over the lane's 16 columns reduced over the D/16
//   lanes of the head; alpha_ji, alpha_ij recomputed from the saved statistics.
#include "gat_args.cuh"

namespace agnn {
namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int K = 128;
// SUB lanes per row, RPW rows per warp, CPL columns (V4 float4) per lane
template <int SUB_>
struct Lay {
  static constexpr int SUB = SUB_, RPW = 32 / SUB, CPL = K / SUB, V4 = CPL / 4;
};

// a lane's V4 x 4-column slice of a feature row, as loaded: fp32 = V4 x 16 B,
// bf16 = V4 / 2 x 16 B (kept packed until use)
template <typename TP, int V4>
struct Cols;
template <int V4>
struct Cols<float, V4> {
  float4 v[V4];
  __device__ __forceinline__ void load(const float* p) {
#pragma unroll
    for (int i = 0; i < V4; ++i) v[i] = ldg4(p + 4 * i);
  }
  __device__ __forceinline__ void load(const float* p, uint64_t pol) {
#pragma unroll
    for (int i = 0; i < V4; ++i) v[i] = ldg4_pol(p + 4 * i, pol);
  }
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int i = 0; i < V4; ++i) v[i] = f4(0.f);
  }
  __device__ __forceinline__ float4 get(int i) const { return v[i]; }
};
template <int V4>
struct Cols<bf16, V4> {
  static_assert(V4 % 2 == 0, "bf16 slices are whole 16-byte loads");
  uint4 v[V4 / 2];
  __device__ __forceinline__ void load(const bf16* p) {
#pragma unroll
    for (int i = 0; i < V4 / 2; ++i) v[i] = __ldg(reinterpret_cast<const uint4*>(p) + i);
  }
  __device__ __forceinline__ void load(const bf16* p, uint64_t pol) {
#pragma unroll
    for (int i = 0; i < V4 / 2; ++i) v[i] = ldg16_pol(reinterpret_cast<const uint4*>(p) + i, pol);
  }
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int i = 0; i < V4 / 2; ++i) v[i] = make_uint4(0u, 0u, 0u, 0u);
  }
  __device__ __forceinline__ float4 get(int i) const {
    const uint4 w = v[i >> 1];
    return (i & 1) ? bf4_to_f4(make_uint2(w.z, w.w)) : bf4_to_f4(make_uint2(w.x, w.y));
  }
};

template <typename TP, int U16>
constexpr int fwd_u() { return sizeof(TP) == 2 ? U16 : 4; }

constexpr int kMaxShort = 32;  // plan short_max <= 64 is clamped to this by the launcher

// Software pipeline over a warp's rows (iteration k = RPW rows): the 16-byte record
// {row, degree, beg} of iteration k+2 and the column ids of iteration k+1 load
// while iteration k computes, so a short row costs one exposed latency (its
// gathers) instead of a chain of four (row id, row_ptr, column ids, gathers).
// Lane q of a row's SUB lanes holds the ids of edges q, q + SUB, ... (CW words).
template <int SUB>
struct RowPipe {
  static constexpr int RPW = 32 / SUB, CW = kMaxShort / SUB;
  const int4* meta;
  const int32_t* col;
  int64_t n;
  int g, q;
  __device__ __forceinline__ int4 rec(int64_t base) const {
    const int64_t r = base + g;
    return r < n ? __ldg(meta + r) : make_int4(0, 0, 0, 0);
  }
  __device__ static __forceinline__ int64_t beg_of(int4 m) {
    return (int64_t)(((uint64_t)(uint32_t)m.w << 32) | (uint64_t)(uint32_t)m.z);
  }
  __device__ __forceinline__ void cols(int4 m, int (&c)[CW]) const {
    const int64_t b = beg_of(m);
#pragma unroll
    for (int k = 0; k < CW; ++k) {
      const int e = q + k * SUB;
      c[k] = e < m.y ? __ldg(col + b + e) : -1;
    }
  }
  // id of edge e of this lane's row, or -1 (e warp-uniform; register selects, no
  // local-memory indexing)
  __device__ __forceinline__ int id(const int (&c)[CW], int e, int lane) const {
    const int w = e / SUB;
    int v = c[0];
#pragma unroll
    for (int k = 1; k < CW; ++k) v = w == k ? c[k] : v;
    return __shfl_sync(0xffffffffu, v, (lane & ~(SUB - 1)) + (e % SUB));
  }
};

// ---------------------------------------------------------------- forward
// QF: also u_i, C_i and Q_i of the factored backward (gat_k128.cu forward, gat_args.cuh)
template <typename TP, int NH, int SUB, int MINB, int U16, bool QF>
__global__ void __launch_bounds__(256, MINB)
gat_fwd_short_kernel(const int4* __restrict__ meta, const int32_t* __restrict__ col,
                     int64_t n_rows, int64_t row_begin, const TP* __restrict__ P,
                     const float* __restrict__ st, float slope, int act, GatFwdOut o,
                     uint32_t col_mask, uint32_t hot_thr, int cold_first) {
  using LY = Lay<SUB>;
  using RP = RowPipe<SUB>;
  constexpr int RPW = LY::RPW, CPL = LY::CPL, V4 = LY::V4, CW = RP::CW;
  constexpr int D = K / NH, U = fwd_u<TP, U16>();
  static_assert(D >= CPL, "a lane's columns lie in one head");
  static_assert(kMaxShort % U == 0, "whole batches");
  const int lane = threadIdx.x & 31, g = lane / SUB, q = lane % SUB;
  const int c0 = q * CPL, h = c0 / D;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t step = nw * RPW;
  const RP rp{meta, col, n_rows, g, q};
  const Gath ga(col_mask, hot_thr, cold_first);
  int64_t base = gw * RPW;
  int4 m_cur = rp.rec(base), m_nxt = rp.rec(base + step);
  int c_cur[CW];
  rp.cols(m_cur, c_cur);
  for (; base < n_rows; base += step) {
    int c_nxt[CW];
    rp.cols(m_nxt, c_nxt);
    const int4 m_nn = rp.rec(base + 2 * step);
    const bool ok = base + g < n_rows;
    const int64_t row = m_cur.x;
    const int deg = min(m_cur.y, kMaxShort);
    const int maxdeg = __reduce_max_sync(FULL, deg);
    const int64_t grow = row_begin + row;
    const float si = ok ? __ldg(st + grow * (2 * NH) + h) : 0.f;
    float m = -INFINITY, l = 0.f, lc = 0.f;
    float4 acc[V4], accu[V4];
#pragma unroll
    for (int v = 0; v < V4; ++v) acc[v] = accu[v] = f4(0.f);
#pragma unroll 1
    for (int b0 = 0; b0 < maxdeg; b0 += U) {
      {
        int j[U];
#pragma unroll
        for (int u = 0; u < U; ++u) j[u] = rp.id(c_cur, b0 + u, lane);
        float tj[U];
        Cols<TP, V4> pj[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (j[u] >= 0) {
            const int64_t jr = ga.row(j[u]);
            const uint64_t pol = ga.policy(j[u]);
            tj[u] = ldg1_pol(st + jr * (2 * NH) + NH + h, pol);
            pj[u].load(P + jr * K + c0, pol);
          } else {
            tj[u] = 0.f;
            pj[u].zero();
          }
        }
        float e[U], pre[U], bm = m;
#pragma unroll
        for (int u = 0; u < U; ++u) {
          pre[u] = si + tj[u];
          e[u] = j[u] >= 0 ? fmaxf(pre[u], slope * pre[u]) : -INFINITY;  // LReLU, 0 <= slope <= 1
          bm = fmaxf(bm, e[u]);
        }
        if (bm != -INFINITY) {  // this row has edges in the batch
          const float sc = ex2(m - bm);  // 0 on the first batch (m = -inf)
          l = __fmul_rn(l, sc);  // never contracted (training and inference variants agree)
          if constexpr (QF) lc = __fmul_rn(lc, sc);
#pragma unroll
          for (int v = 0; v < V4; ++v) {
            acc[v] = mul4(sc, acc[v]);
            if constexpr (QF) accu[v] = mul4(sc, accu[v]);
          }
          m = bm;
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const float p = ex2(e[u] - m);  // 0 for padding edges
            l = __fadd_rn(l, p);
            const float pc = pre[u] > 0.f ? p : p * slope;
            if constexpr (QF) lc = __fadd_rn(lc, pc);
#pragma unroll
            for (int v = 0; v < V4; ++v) {
              const float4 x = pj[u].get(v);
              acc[v] = fma4(p, x, acc[v]);
              if constexpr (QF) accu[v] = fma4(pc, x, accu[v]);
            }
          }
        }
      }
    }
    if (ok) {
      const float inv = l > 0.f ? 1.f / l : 0.f;
      const float r = l > 0.f ? lc / l : 0.f;
#pragma unroll
      for (int v = 0; v < V4; ++v) {
        const float4 z = mul4(inv, acc[v]);
        if (o.Z) st4(o.Z + row * K + c0 + 4 * v, z);
        st4(o.Hout + row * K + c0 + 4 * v, act_fwd4(act, z));
        if constexpr (QF) st4(o.Q + row * K + c0 + 4 * v, mul4(inv, fma4(-r, acc[v], accu[v])));
      }
      if (o.m && (c0 % D) == 0) {
        o.m[row * NH + h] = l > 0.f ? m : 0.f;
        o.l[row * NH + h] = l;
      }
    }
    m_cur = m_nxt;
    m_nxt = m_nn;
#pragma unroll
    for (int k = 0; k < CW; ++k) c_cur[k] = c_nxt[k];
  }
}

// ---------------------------------------------------------------- backward
template <typename TP>
__device__ __forceinline__ const TP* pick_rows(const float* f, const bf16* h);
template <>
__device__ __forceinline__ const float* pick_rows<float>(const float* f, const bf16*) { return f; }
template <>
__device__ __forceinline__ const bf16* pick_rows<bf16>(const float*, const bf16* h) { return h; }

template <typename TP, int NH, int SUB, int U, int MINB>
__global__ void __launch_bounds__(256, MINB)
gat_bwd_short_kernel(const int4* __restrict__ meta, const int32_t* __restrict__ col,
                     int64_t n_rows, int64_t row_begin, GatBwdArgs A, int64_t da_row0,
                     uint32_t col_mask, uint32_t hot_thr, int cold_first) {
  using LY = Lay<SUB>;
  using RP = RowPipe<SUB>;
  constexpr int RPW = LY::RPW, CPL = LY::CPL, V4 = LY::V4, CW = RP::CW;
  constexpr int D = K / NH, HLS = D / CPL;  // HLS lanes share a head
  static_assert(D >= CPL, "a lane's columns lie in one head");
  static_assert(kMaxShort % U == 0, "whole batches");
  const int lane = threadIdx.x & 31, g = lane / SUB, q = lane % SUB;
  const int c0 = q * CPL, h = c0 / D;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t step = nw * RPW;
  const TP* Pb = pick_rows<TP>(A.P, A.P16);
  const TP* Gb = pick_rows<TP>(A.G, A.G16);
  const float slope = A.slope;
  const RP rp{meta, col, n_rows, g, q};
  const Gath ga(col_mask, hot_thr, cold_first);
  float4 da1[V4], da2[V4];
#pragma unroll
  for (int v = 0; v < V4; ++v) da1[v] = da2[v] = f4(0.f);
  int64_t base = gw * RPW;
  int4 m_cur = rp.rec(base), m_nxt = rp.rec(base + step);
  int c_cur[CW];
  rp.cols(m_cur, c_cur);
  for (; base < n_rows; base += step) {
    int c_nxt[CW];
    rp.cols(m_nxt, c_nxt);
    const int4 m_nn = rp.rec(base + 2 * step);
    const bool ok = base + g < n_rows;
    const int64_t row = m_cur.x;
    const int deg = min(m_cur.y, kMaxShort);
    const int maxdeg = __reduce_max_sync(FULL, deg);  // warp-uniform trip count (shuffles inside)
    const int64_t grow = row_begin + row;
    float4 Pj[V4], Gj[V4];
    {
      Cols<TP, V4> cp, cg;
      cp.load(Pb + grow * K + c0);
      cg.load(Gb + grow * K + c0);
#pragma unroll
      for (int v = 0; v < V4; ++v) {
        Pj[v] = cp.get(v);
        Gj[v] = cg.get(v);
      }
    }
    const float4 rj = __ldg(A.rec + grow * NH + h);  // {s_j, m_j, 1/l_j, delta_j}
    const float tj = __ldg(A.st + grow * (2 * NH) + NH + h);
    float4 acc[V4];
#pragma unroll
    for (int v = 0; v < V4; ++v) acc[v] = f4(0.f);
    float ds = 0.f, dt = 0.f;
#pragma unroll 1
    for (int b0 = 0; b0 < maxdeg; b0 += U) {
      {
        int i[U];
#pragma unroll
        for (int u = 0; u < U; ++u) i[u] = rp.id(c_cur, b0 + u, lane);
        Cols<TP, V4> pi[U], gi[U];
        float4 ri[U];
        float ti[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (i[u] >= 0) {
            const int64_t ir = ga.row(i[u]);
            const uint64_t pol = ga.policy(i[u]);
            pi[u].load(Pb + ir * K + c0, pol);
            gi[u].load(Gb + ir * K + c0, pol);
            ri[u] = ldg4_pol(reinterpret_cast<const float*>(A.rec + ir * NH + h), pol);
            ti[u] = ldg1_pol(A.st + ir * (2 * NH) + NH + h, pol);
          } else {
            pi[u].zero();
            gi[u].zero();
            ri[u] = f4(0.f);
            ti[u] = 0.f;
          }
        }
        float x1[U], x2[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          float a = 0.f, b = 0.f;
#pragma unroll
          for (int v = 0; v < V4; ++v) {
            a += dot4(Gj[v], pi[u].get(v));  // G_j . P_i  (row role)
            b += dot4(gi[u].get(v), Pj[v]);  // G_i . P_j  (column role)
          }
          x1[u] = a;
          x2[u] = b;
        }
#pragma unroll
        for (int o = 1; o < HLS; o <<= 1) {
#pragma unroll
          for (int u = 0; u < U; ++u) {
            x1[u] += __shfl_xor_sync(FULL, x1[u], o);
            x2[u] += __shfl_xor_sync(FULL, x2[u], o);
          }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const bool vm = i[u] >= 0;
          // row role: entry (j,i) of row j
          const float pre = rj.x + ti[u];
          const float e = fmaxf(pre, slope * pre);
          const float aji = ex2(e - rj.y) * rj.z;
          const float dcji = aji * (pre > 0.f ? 1.f : slope) * (x1[u] - rj.w);
          // column role: entry (i,j) of row i
          const float pre2 = ri[u].x + tj;
          const float e2 = fmaxf(pre2, slope * pre2);
          const float aij = ex2(e2 - ri[u].y) * ri[u].z;
          const float dcij = aij * (pre2 > 0.f ? 1.f : slope) * (x2[u] - ri[u].w);
          if (vm) {
            ds += dcji;
            dt += dcij;
#pragma unroll
            for (int v = 0; v < V4; ++v) acc[v] = fma4(aij, gi[u].get(v), acc[v]);
          }
        }
      }
    }
    if (ok) {
#pragma unroll
      for (int v = 0; v < V4; ++v) {
        const int cc = (c0 % D) + 4 * v;
        const float4 a1v = ldg4(A.a + h * 2 * D + cc);
        const float4 a2v = ldg4(A.a + h * 2 * D + D + cc);
        float4 dp = fma4(ds, a1v, acc[v]);
        dp = fma4(dt, a2v, dp);
        st4(A.dP + row * K + c0 + 4 * v, dp);
        da1[v] = fma4(ds, Pj[v], da1[v]);
        da2[v] = fma4(dt, Pj[v], da2[v]);
      }
    }
    m_cur = m_nxt;
    m_nxt = m_nn;
#pragma unroll
    for (int k = 0; k < CW; ++k) c_cur[k] = c_nxt[k];
  }
  // the RPW row slots of the warp hold the same columns: fold them (fixed order), then
  // the first slot writes the warp's da partial row
#pragma unroll
  for (int o = SUB; o < 32; o <<= 1) {
#pragma unroll
    for (int v = 0; v < V4; ++v) {
      da1[v].x += __shfl_xor_sync(FULL, da1[v].x, o);
      da1[v].y += __shfl_xor_sync(FULL, da1[v].y, o);
      da1[v].z += __shfl_xor_sync(FULL, da1[v].z, o);
      da1[v].w += __shfl_xor_sync(FULL, da1[v].w, o);
      da2[v].x += __shfl_xor_sync(FULL, da2[v].x, o);
      da2[v].y += __shfl_xor_sync(FULL, da2[v].y, o);
      da2[v].z += __shfl_xor_sync(FULL, da2[v].z, o);
      da2[v].w += __shfl_xor_sync(FULL, da2[v].w, o);
    }
  }
  if (g == 0) {
#pragma unroll
    for (int v = 0; v < V4; ++v) {
      st4(A.da_part + (da_row0 + gw) * 2 * K + c0 + 4 * v, da1[v]);
      st4(A.da_part + (da_row0 + gw) * 2 * K + K + c0 + 4 * v, da2[v]);
    }
  }
}

// factored backward (column role only; ds_j from the prologue, gat_args.cuh): per
// edge the lane gathers its slice of G_i and the record of its head, recomputes
// alpha_ij, c'_ij = alpha_ij lambda_ij, and accumulates acc += alpha G_i, v += c' G_i,
// sd += c' delta_i (every lane of a head the same scalars); per row
// dt_j = P_j . v_j - sd, dP_j = acc + ds_j a1 + dt_j a2.
template <typename TP, int NH, int SUB, int U, int MINB>
__global__ void __launch_bounds__(256, MINB)
gat_bwd_short_f_kernel(const int4* __restrict__ meta, const int32_t* __restrict__ col,
                       int64_t n_rows, int64_t row_begin, GatBwdArgs A, int64_t da_row0,
                       uint32_t col_mask, uint32_t hot_thr, int cold_first) {
  using LY = Lay<SUB>;
  using RP = RowPipe<SUB>;
  constexpr int CPL = LY::CPL, V4 = LY::V4, CW = RP::CW;
  constexpr int D = K / NH, HLS = D / CPL;  // HLS lanes share a head
  static_assert(D >= CPL, "a lane's columns lie in one head");
  static_assert(kMaxShort % U == 0, "whole batches");
  const int lane = threadIdx.x & 31, g = lane / SUB, q = lane % SUB;
  const int c0 = q * CPL, h = c0 / D;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t step = nw * LY::RPW;
  const TP* Pb = pick_rows<TP>(A.P, A.P16);
  const TP* Gb = pick_rows<TP>(A.G, A.G16);
  const float slope = A.slope;
  const RP rp{meta, col, n_rows, g, q};
  const Gath ga(col_mask, hot_thr, cold_first);
  float4 da1[V4], da2[V4];
#pragma unroll
  for (int v = 0; v < V4; ++v) da1[v] = da2[v] = f4(0.f);
  int64_t base = gw * LY::RPW;
  int4 m_cur = rp.rec(base), m_nxt = rp.rec(base + step);
  int c_cur[CW];
  rp.cols(m_cur, c_cur);
  for (; base < n_rows; base += step) {
    int c_nxt[CW];
    rp.cols(m_nxt, c_nxt);
    const int4 m_nn = rp.rec(base + 2 * step);
    const bool ok = base + g < n_rows;
    const int64_t row = m_cur.x;
    const int deg = min(m_cur.y, kMaxShort);
    const int maxdeg = __reduce_max_sync(FULL, deg);  // warp-uniform trip count
    const int64_t grow = row_begin + row;
    const float tj = __ldg(A.st + grow * (2 * NH) + NH + h);
    float4 acc[V4], accv[V4];
#pragma unroll
    for (int v = 0; v < V4; ++v) acc[v] = accv[v] = f4(0.f);
    float sd = 0.f;
#pragma unroll 1
    for (int b0 = 0; b0 < maxdeg; b0 += U) {
      int i[U];
#pragma unroll
      for (int u = 0; u < U; ++u) i[u] = rp.id(c_cur, b0 + u, lane);
      Cols<TP, V4> gi[U];
      float4 ri[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (i[u] >= 0) {
          const int64_t ir = ga.row(i[u]);
          const uint64_t pol = ga.policy(i[u]);
          gi[u].load(Gb + ir * K + c0, pol);
          ri[u] = ldg4_pol(reinterpret_cast<const float*>(A.rec + ir * NH + h), pol);
        } else {
          gi[u].zero();
          ri[u] = f4(0.f);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (i[u] >= 0) {
          const float pre = ri[u].x + tj;
          const float e = fmaxf(pre, slope * pre);
          const float al = ex2(e - ri[u].y) * ri[u].z;
          const float cc = pre > 0.f ? al : al * slope;
          sd = fmaf(cc, ri[u].w, sd);
#pragma unroll
          for (int v = 0; v < V4; ++v) {
            const float4 x = gi[u].get(v);
            acc[v] = fma4(al, x, acc[v]);
            accv[v] = fma4(cc, x, accv[v]);
          }
        }
      }
    }
    float4 Pj[V4];
    {
      Cols<TP, V4> cp;
      cp.load(Pb + grow * K + c0);
#pragma unroll
      for (int v = 0; v < V4; ++v) Pj[v] = cp.get(v);
    }
    float x = 0.f;
#pragma unroll
    for (int v = 0; v < V4; ++v) x += dot4(Pj[v], accv[v]);
#pragma unroll
    for (int o = 1; o < HLS; o <<= 1) x += __shfl_xor_sync(FULL, x, o);
    if (ok) {
      const float dt = x - sd;
      const float ds = A.ds_row[row * NH + h];
#pragma unroll
      for (int v = 0; v < V4; ++v) {
        const int cc = (c0 % D) + 4 * v;
        const float4 a1v = ldg4(A.a + h * 2 * D + cc);
        const float4 a2v = ldg4(A.a + h * 2 * D + D + cc);
        float4 dp = fma4(ds, a1v, acc[v]);
        dp = fma4(dt, a2v, dp);
        st4(A.dP + row * K + c0 + 4 * v, dp);
        da1[v] = fma4(ds, Pj[v], da1[v]);
        da2[v] = fma4(dt, Pj[v], da2[v]);
      }
    }
    m_cur = m_nxt;
    m_nxt = m_nn;
#pragma unroll
    for (int k = 0; k < CW; ++k) c_cur[k] = c_nxt[k];
  }
#pragma unroll
  for (int o = SUB; o < 32; o <<= 1) {
#pragma unroll
    for (int v = 0; v < V4; ++v) {
      da1[v].x += __shfl_xor_sync(FULL, da1[v].x, o);
      da1[v].y += __shfl_xor_sync(FULL, da1[v].y, o);
      da1[v].z += __shfl_xor_sync(FULL, da1[v].z, o);
      da1[v].w += __shfl_xor_sync(FULL, da1[v].w, o);
      da2[v].x += __shfl_xor_sync(FULL, da2[v].x, o);
      da2[v].y += __shfl_xor_sync(FULL, da2[v].y, o);
      da2[v].z += __shfl_xor_sync(FULL, da2[v].z, o);
      da2[v].w += __shfl_xor_sync(FULL, da2[v].w, o);
    }
  }
  if (g == 0) {
#pragma unroll
    for (int v = 0; v < V4; ++v) {
      st4(A.da_part + (da_row0 + gw) * 2 * K + c0 + 4 * v, da1[v]);
      st4(A.da_part + (da_row0 + gw) * 2 * K + K + c0 + 4 * v, da2[v]);
    }
  }
}

template <typename F>
int grid_for(F* f) {
  return persistent_blocks(reinterpret_cast<const void*>(f));
}

}  // namespace

#define AGNN_SHORT_DISPATCH(NH_, CALL)                                  \
  do {                                                                  \
    if (NH_ == 1) { constexpr int NH = 1; CALL; }                       \
    else if (NH_ == 2) { constexpr int NH = 2; CALL; }                  \
    else if (NH_ == 4) { constexpr int NH = 4; CALL; }                  \
    else if (NH_ == 8) { constexpr int NH = 8; CALL; }                  \
    else return fail(AGNN_EUNSUPPORTED, "GAT k'=128: heads must be 1/2/4/8"); \
  } while (0)

template <typename TP>
agnn_status gat_fwd_short(const Items& it, int heads, const TP* P, const float* st, float slope,
                          int act, const GatFwdOut& o, cudaStream_t s) {
  if (it.n_short == 0) return AGNN_OK;
  AGNN_SHORT_DISPATCH(heads, ({
    // fp32: 8 lanes per row, 2 blocks / SM (the 3-block variant spills); bf16: 16 lanes
    // per row, 3 blocks / SM, 4-edge batches (measured C5, round 1)
    using KF = void (*)(const int4*, const int32_t*, int64_t, int64_t, const TP*, const float*,
                        float, int, GatFwdOut, uint32_t, uint32_t, int);
    KF kern;
    if (sizeof(TP) == 2)
      kern = o.Q ? (KF)gat_fwd_short_kernel<TP, NH, 16, 3, 4, true>
                 : (KF)gat_fwd_short_kernel<TP, NH, 16, 3, 4, false>;
    else
      kern = o.Q ? (KF)gat_fwd_short_kernel<TP, NH, 8, 2, 8, true>
                 : (KF)gat_fwd_short_kernel<TP, NH, 8, 2, 8, false>;
    kern<<<grid_for(kern), 256, 0, s>>>(it.short_meta, it.col, it.n_short, it.row_begin, P, st,
                                         slope, act, o, it.col_mask, it.hot_thr, it.cold_first);
    AGNN_LAUNCH_CHECK("gat_fwd_short_kernel");
  }));
  return AGNN_OK;
}
template agnn_status gat_fwd_short<float>(const Items&, int, const float*, const float*, float, int,
                                          const GatFwdOut&, cudaStream_t);
template agnn_status gat_fwd_short<bf16>(const Items&, int, const bf16*, const float*, float, int,
                                         const GatFwdOut&, cudaStream_t);

agnn_status gat_bwd_short(const Items& it, int heads, const GatBwdArgs& A, int64_t da_row0,
                          int64_t* warps, cudaStream_t s) {
  *warps = 0;
  if (it.n_short == 0) return AGNN_OK;
  AGNN_SHORT_DISPATCH(heads, ({
    int grid;
    // one 8-warp block per SM with up to 255 registers: U edges x 4 rows of gathers
    // in flight per warp without spilling (bf16 rows are half the registers)
    if (A.P16) {
      auto launch = [&](auto* kern) {
        grid = grid_for(kern);
        kern<<<grid, 256, 0, s>>>(it.short_meta, it.col, it.n_short, it.row_begin, A, da_row0,
                                  it.col_mask, it.hot_thr, it.cold_first);
      };
      launch(gat_bwd_short_kernel<bf16, NH, 16, 4, 2>);
    } else {
      auto* kern = gat_bwd_short_kernel<float, NH, 16, 2, 2>;
      grid = grid_for(kern);
      kern<<<grid, 256, 0, s>>>(it.short_meta, it.col, it.n_short, it.row_begin, A, da_row0,
                                it.col_mask, it.hot_thr, it.cold_first);
    }
    AGNN_LAUNCH_CHECK("gat_bwd_short_kernel");
    *warps = (int64_t)grid * 8;
  }));
  return AGNN_OK;
}

agnn_status gat_bwd_short_f(const Items& it, int heads, const GatBwdArgs& A, int64_t da_row0,
                            int64_t* warps, cudaStream_t s) {
  *warps = 0;
  if (it.n_short == 0) return AGNN_OK;
  AGNN_SHORT_DISPATCH(heads, ({
    // 16 lanes per row (2 rows per warp), 2-edge fp32 / 4-edge bf16 batches, 3 blocks /
    // SM (measured C5, round 1: 14.7 -> 13.5 ms fp32 against 4-edge batches at 2 / SM)
    using KB = void (*)(const int4*, const int32_t*, int64_t, int64_t, GatBwdArgs, int64_t,
                        uint32_t, uint32_t, int);
    KB kern = A.P16 ? (KB)gat_bwd_short_f_kernel<bf16, NH, 16, 4, 3>
                    : (KB)gat_bwd_short_f_kernel<float, NH, 16, 2, 3>;
    const int grid = grid_for(kern);
    kern<<<grid, 256, 0, s>>>(it.short_meta, it.col, it.n_short, it.row_begin, A, da_row0,
                              it.col_mask, it.hot_thr, it.cold_first);
    AGNN_LAUNCH_CHECK("gat_bwd_short_kernel");
    *warps = (int64_t)grid * 8;
  }));
  return AGNN_OK;
}

}  // namespace agnn
