// gat_bundle.cu — GAT k' = 128 sparse kernels for BUNDLES of short rows.
//
// Same arithmetic as gat_k128.cu / gat_short.cu (PAPER.md:177 forward with the
// graph softmax of :191; the factored backward of gat_args.cuh for :250-254),
// different work decomposition.  A Kronecker graph has most of its rows short
// (S§8(d): median degree 2-3) and a warp-per-row kernel pays a chain of
// dependent loads and one exposed gather latency per row.  Here the plan packs
// consecutive short rows into bundles of at most 32 stored entries
// (plan.cu), and a warp processes one bundle exactly like one 32-edge batch of
// the long-row kernels: lane e owns stored entry e (scores, segmented softmax
// reductions over the lanes of its row), then the warp walks the entries with
// the gathered rows of the next group in flight and finishes each row at its
// last entry.  The bundle records, row records and column ids of the next
// bundles load while the current bundle is processed.
//
// Row maxima and sums are exact segmented reductions over a row's lanes (a
// bundle holds whole rows, so no online rescaling is needed); the order is
// fixed, so results are deterministic and the training (QF) and inference
// variants agree bitwise.
#include "gat_args.cuh"

namespace agnn {
namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int K = 128;

template <typename TP>
__device__ __forceinline__ const TP* pick_tp(const float* f, const bf16* h);
template <>
__device__ __forceinline__ const float* pick_tp<float>(const float* f, const bf16*) { return f; }
template <>
__device__ __forceinline__ const bf16* pick_tp<bf16>(const float*, const bf16* h) { return h; }

// gathered rows per prefetch group: 4 for both storage types — the row finish is
// inlined after every entry of the unrolled group loop, and 8-row bf16 groups
// (16 copies) overflowed the instruction cache (measured: bf16 forward 10 -> 28 ms)
template <typename TP>
constexpr int group_rows() { return 4; }

// inclusive segmented scans over the lanes of one row (key = row slot; rows are
// contiguous lane ranges, so equal keys at distance o mean the same row)
__device__ __forceinline__ float seg_max(float v, int key, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const float u = __shfl_up_sync(FULL, v, o);
    const int k = __shfl_up_sync(FULL, key, o);
    if (lane >= o && k == key) v = fmaxf(v, u);
  }
  return v;
}
__device__ __forceinline__ float seg_sum(float v, int key, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const float u = __shfl_up_sync(FULL, v, o);
    const int k = __shfl_up_sync(FULL, key, o);
    if (lane >= o && k == key) v = __fadd_rn(v, u);
  }
  return v;
}

// One bundle as seen by the lanes of a warp.
template <int NH>
struct BMap {
  int4 B;        // {first short record, rows, entries, 0} (uniform)
  int4 meta;     // lane r < rows: {row, degree, beg lo, beg hi}
  uint32_t starts;  // bit e set: entry e is the first of its row (uniform)
  int rs;        // lane e < entries: row slot of entry e (else -1)
  int last;      // lane e: last entry of its row
  int c;         // lane e: column entry (with the L2 class bits)
  float sc[NH];  // lane r: per-head scalars of row r (st + soff)
  float tj[NH];  // lane e: t_j of its column (forward; loaded a bundle ahead)
};

template <int NH, bool TJ = false>
__device__ __forceinline__ void bmap(BMap<NH>& m, int4 B, int4 meta, const int32_t* __restrict__ col,
                                     const float* __restrict__ st, int64_t row_begin, int soff,
                                     int lane, const Gath* ga = nullptr) {
  m.B = B;
  m.meta = meta;
  const bool isrow = lane < B.y;
  const int deg = isrow ? meta.y : 0;
  int incl = deg;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int t = __shfl_up_sync(FULL, incl, o);
    if (lane >= o) incl += t;
  }
  const int off = incl - deg;
  m.starts = __reduce_or_sync(FULL, isrow ? (1u << off) : 0u);
  const bool valid = lane < B.z;
  const uint32_t upto = lane == 31 ? FULL : ((2u << lane) - 1u);
  m.rs = valid ? __popc(m.starts & upto) - 1 : -1;
  const int src = valid ? m.rs : 0;
  const int64_t beg = (int64_t)(((uint64_t)(uint32_t)__shfl_sync(FULL, meta.w, src) << 32) |
                                (uint64_t)(uint32_t)__shfl_sync(FULL, meta.z, src));
  const int offr = __shfl_sync(FULL, off, src), degr = __shfl_sync(FULL, deg, src);
  m.last = offr + degr - 1;
  m.c = valid ? __ldg(col + beg + (lane - offr)) : 0;
#pragma unroll
  for (int h = 0; h < NH; ++h)
    m.sc[h] = isrow ? __ldg(st + (row_begin + meta.x) * (2 * NH) + soff + h) : 0.f;
  if constexpr (TJ) {  // the entries' t_j (the forward's scores), one bundle ahead
    const float* tp = st + ga->row(m.c) * (2 * NH) + NH;
    const uint64_t pol = ga->policy(m.c);
#pragma unroll
    for (int h = 0; h < NH; ++h) m.tj[h] = valid ? ldg1_pol(tp + h, pol) : 0.f;
  }
}

__device__ __forceinline__ int4 ld_rec(const int4* p, int64_t i, int64_t n) {
  return i < n ? __ldg(p + i) : make_int4(0, 0, 0, 0);
}

// ---------------------------------------------------------------- forward
template <typename TP, int NH, bool QF, int MINB>
__global__ void __launch_bounds__(256, MINB)
gat_fwd_bundle_kernel(Items it, const TP* __restrict__ P, const float* __restrict__ st, float slope,
                      int act, GatFwdOut o) {
  constexpr int D = K / NH, HL = D / 4, GR = group_rows<TP>();
  __shared__ float sPw[QF ? 1 : 8][NH][33];
  __shared__ float2 sP2[QF ? 8 : 1][NH][33];
  __shared__ float2 sSt[8][32][NH];  // row slot, head: {l, lc}
  __shared__ float sM[8][32][NH];    // row slot, head: row maximum
  __shared__ int sJ[8][32];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int hv = lane / HL, cq = lane * 4;
  const int64_t nb = it.n_bundles;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const Gath ga(it);
  using SL = Slice<TP>;
  // pipeline: the current bundle mapped (column ids in flight), the next bundle's
  // row records loaded, the bundle record after it loaded
  BMap<NH> cur;
  {
    const int4 B0 = ld_rec(it.bundles, gw, nb);
    bmap<NH, true>(cur, B0, lane < B0.y ? __ldg(it.short_meta + B0.x + lane) : make_int4(0, 0, 0, 0),
                   it.col, st, it.row_begin, 0, lane, &ga);
  }
  int4 Bn = ld_rec(it.bundles, gw + nw, nb);
  int4 Mn = lane < Bn.y ? __ldg(it.short_meta + Bn.x + lane) : make_int4(0, 0, 0, 0);
  int4 Bnn = ld_rec(it.bundles, gw + 2 * nw, nb);
  for (int64_t b = gw; b < nb; b += nw) {
    BMap<NH> nxt;
    bmap<NH, true>(nxt, Bn, Mn, it.col, st, it.row_begin, 0, lane, &ga);
    Mn = lane < Bnn.y ? __ldg(it.short_meta + Bnn.x + lane) : make_int4(0, 0, 0, 0);
    Bn = Bnn;
    Bnn = ld_rec(it.bundles, b + 3 * nw, nb);

    const int ne = cur.B.z;
    const bool valid = lane < ne;
    const int c = cur.c, rs = cur.rs;
    sJ[wib][lane] = c;
    __syncwarp();
    typename SL::raw qa[GR], qb[GR];
#pragma unroll
    for (int u = 0; u < GR; ++u)
      qa[u] = u < ne ? SL::load(P + ga.row(sJ[wib][u]) * K + cq, ga.policy(sJ[wib][u])) : SL::zero();
    const float* tj = cur.tj;  // loaded a bundle ahead (bmap)
    const int src = valid ? rs : 0;
#pragma unroll
    for (int h = 0; h < NH; ++h) {
      const float pre = __shfl_sync(FULL, cur.sc[h], src) + tj[h];
      const float e = valid ? fmaxf(pre, slope * pre) : -INFINITY;  // LReLU, 0 <= slope <= 1
      const float mrow = __shfl_sync(FULL, seg_max(e, rs, lane), valid ? cur.last : lane);
      const float p = valid ? ex2(e - mrow) : 0.f;
      const float l = __shfl_sync(FULL, seg_sum(p, rs, lane), valid ? cur.last : lane);
      float lc = 0.f;
      if constexpr (QF) {
        const float pc = pre > 0.f ? p : p * slope;
        lc = __shfl_sync(FULL, seg_sum(pc, rs, lane), valid ? cur.last : lane);
        sP2[wib][h][lane] = make_float2(p, pc);
      } else {
        sPw[wib][h][lane] = p;
      }
      if (valid && lane == cur.last) {
        sSt[wib][rs][h] = make_float2(l, lc);
        sM[wib][rs][h] = mrow;
      }
    }
    const uint32_t ends = __ballot_sync(FULL, valid && lane == cur.last);
    __syncwarp();
    float4 acc = f4(0.f), accu = f4(0.f);
    auto edge = [&](int e, const typename SL::raw& r) {
      const float4 x = SL::f(r);
      if constexpr (QF) {
        const float2 pw = sP2[wib][hv][e];
        acc = fma4(pw.x, x, acc);
        accu = fma4(pw.y, x, accu);
      } else {
        acc = fma4(sPw[wib][hv][e], x, acc);
      }
      if ((ends >> e) & 1u) {  // last entry of its row: finish the row
        const int slot = __popc(cur.starts & (e == 31 ? FULL : ((2u << e) - 1u))) - 1;
        const int64_t row = __shfl_sync(FULL, cur.meta.x, slot);
        const float2 sv = sSt[wib][slot][hv];
        const float inv = sv.x > 0.f ? 1.f / sv.x : 0.f;
        const float4 z = mul4(inv, acc);
        if (o.Z) st4(o.Z + row * K + cq, z);
        st4(o.Hout + row * K + cq, act_fwd4(act, z));
        if constexpr (QF) {
          const float r = sv.x > 0.f ? sv.y / sv.x : 0.f;
          st4(o.Q + row * K + cq, mul4(inv, fma4(-r, acc, accu)));
        }
        if (o.m && lane < NH) {
          const float ll = sSt[wib][slot][lane].x;
          o.m[row * NH + lane] = ll > 0.f ? sM[wib][slot][lane] : 0.f;
          o.l[row * NH + lane] = ll;
        }
        acc = accu = f4(0.f);
      }
    };
    const TP* Pl = P + cq;
#pragma unroll 1
    for (int g0 = 0; g0 < ne; g0 += 2 * GR) {
#pragma unroll
      for (int u = 0; u < GR; ++u) {
        const int e = g0 + GR + u;
        qb[u] = e < ne ? SL::load(Pl + ga.row(sJ[wib][e]) * K, ga.policy(sJ[wib][e])) : SL::zero();
      }
#pragma unroll
      for (int u = 0; u < GR; ++u)
        if (g0 + u < ne) edge(g0 + u, qa[u]);
#pragma unroll
      for (int u = 0; u < GR; ++u) {
        const int e = g0 + 2 * GR + u;
        qa[u] = e < ne ? SL::load(Pl + ga.row(sJ[wib][e < 32 ? e : 0]) * K,
                                  ga.policy(sJ[wib][e < 32 ? e : 0]))
                       : SL::zero();
      }
#pragma unroll
      for (int u = 0; u < GR; ++u)
        if (g0 + GR + u < ne) edge(g0 + GR + u, qb[u]);
    }
    __syncwarp();
    cur = nxt;
  }
}

// ---------------------------------------------------------------- backward (factored)
// Column role only (ds_j from the prologue): lane e recomputes alpha_ij, c'_ij of
// its entry from rec_i, the row's t_j; segmented sum of c'_ij delta_i per head;
// then acc_j += alpha G_i, v_j += c' G_i over the row's entries and, at its last
// entry, dt_j = P_j . v_j - sum c' delta, dP_j = acc + ds a1 + dt a2.
template <typename TP, int NH, int MINB>
__global__ void __launch_bounds__(256, MINB)
gat_bwd_bundle_kernel(Items it, GatBwdArgs A, int64_t da_row0) {
  constexpr int D = K / NH, HL = D / 4, GR = group_rows<TP>();
  __shared__ float2 sAC[8][NH][33];  // {alpha_ij, c'_ij}
  __shared__ float2 sSt[8][32][NH];  // row slot, head: {sum c' delta, ds}
  __shared__ int sJ[8][32];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  const int hv = lane / HL, cq = lane * 4;
  const int64_t nb = it.n_bundles;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const Gath ga(it);
  using SL = Slice<TP>;
  const TP* Pb = pick_tp<TP>(A.P, A.P16);
  const TP* Gb = pick_tp<TP>(A.G, A.G16);
  const float slope = A.slope;
  const float4 a1v = ldg4(A.a + hv * 2 * D + cq % D);
  const float4 a2v = ldg4(A.a + hv * 2 * D + D + cq % D);
  float4 da1 = f4(0.f), da2 = f4(0.f);
  BMap<NH> cur;
  {
    const int4 B0 = ld_rec(it.bundles, gw, nb);
    bmap(cur, B0, lane < B0.y ? __ldg(it.short_meta + B0.x + lane) : make_int4(0, 0, 0, 0), it.col,
         A.st, it.row_begin, NH, lane);
  }
  int4 Bn = ld_rec(it.bundles, gw + nw, nb);
  int4 Mn = lane < Bn.y ? __ldg(it.short_meta + Bn.x + lane) : make_int4(0, 0, 0, 0);
  int4 Bnn = ld_rec(it.bundles, gw + 2 * nw, nb);
  for (int64_t b = gw; b < nb; b += nw) {
    BMap<NH> nxt;
    bmap(nxt, Bn, Mn, it.col, A.st, it.row_begin, NH, lane);
    Mn = lane < Bnn.y ? __ldg(it.short_meta + Bnn.x + lane) : make_int4(0, 0, 0, 0);
    Bn = Bnn;
    Bnn = ld_rec(it.bundles, b + 3 * nw, nb);

    const int ne = cur.B.z, nr = cur.B.y;
    const bool valid = lane < ne;
    const int c = cur.c, rs = cur.rs;
    sJ[wib][lane] = c;
    // ds_j of the bundle's rows (prologue), row lanes
    float dsr[NH];
#pragma unroll
    for (int h = 0; h < NH; ++h) dsr[h] = lane < nr ? __ldg(A.ds_row + (int64_t)cur.meta.x * NH + h) : 0.f;
    __syncwarp();
    typename SL::raw qa[GR], qb[GR];
#pragma unroll
    for (int u = 0; u < GR; ++u)
      qa[u] = u < ne ? SL::load(Gb + ga.row(sJ[wib][u]) * K + cq, ga.policy(sJ[wib][u])) : SL::zero();
    // P_j of the first two rows (ring of two, refilled two rows ahead)
    float4 pr0 = nr > 0 ? SL::f(SL::load(Pb + ((int64_t)__shfl_sync(FULL, cur.meta.x, 0) + it.row_begin) * K + cq))
                        : f4(0.f);
    float4 pr1 = nr > 1 ? SL::f(SL::load(Pb + ((int64_t)__shfl_sync(FULL, cur.meta.x, 1) + it.row_begin) * K + cq))
                        : f4(0.f);
    {
      const int64_t ir = ga.row(c);
      const uint64_t pol = ga.policy(c);
      const int src = valid ? rs : 0;
#pragma unroll
      for (int h = 0; h < NH; ++h) {
        const float4 r = valid ? ldg4_pol(reinterpret_cast<const float*>(A.rec + ir * NH + h), pol)
                               : f4(0.f);  // {s_i, m_i, 1/l_i, delta_i}
        const float pre = r.x + __shfl_sync(FULL, cur.sc[h], src);
        const float e = fmaxf(pre, slope * pre);
        const float al = valid ? ex2(e - r.y) * r.z : 0.f;
        const float cc = pre > 0.f ? al : al * slope;
        const float sd = __shfl_sync(FULL, seg_sum(cc * r.w, rs, lane), valid ? cur.last : lane);
        const float ds = __shfl_sync(FULL, dsr[h], src);
        sAC[wib][h][lane] = make_float2(al, cc);
        if (valid && lane == cur.last) sSt[wib][rs][h] = make_float2(sd, ds);
      }
    }
    const uint32_t ends = __ballot_sync(FULL, valid && lane == cur.last);
    __syncwarp();
    float4 acc = f4(0.f), accv = f4(0.f);
    auto edge = [&](int e, const typename SL::raw& r) {
      const float4 x = SL::f(r);
      const float2 ac = sAC[wib][hv][e];
      acc = fma4(ac.x, x, acc);
      accv = fma4(ac.y, x, accv);
      if ((ends >> e) & 1u) {
        const int slot = __popc(cur.starts & (e == 31 ? FULL : ((2u << e) - 1u))) - 1;
        const int64_t row = __shfl_sync(FULL, cur.meta.x, slot);
        const float4 Pj = (slot & 1) ? pr1 : pr0;
        if (slot + 2 < nr) {  // refill the ring slot two rows ahead
          // (the load writes its slot directly: a select on the loaded value would
          // wait for it here — ncu r02: 13 % of the kernel's stall samples)
          const TP* pp = Pb + ((int64_t)__shfl_sync(FULL, cur.meta.x, slot + 2) + it.row_begin) * K + cq;
          if (slot & 1) pr1 = SL::f(SL::load(pp));
          else pr0 = SL::f(SL::load(pp));
        }
        float x2 = dot4(Pj, accv);
#pragma unroll
        for (int o = 1; o < HL; o <<= 1) x2 += __shfl_xor_sync(FULL, x2, o);
        const float2 sv = sSt[wib][slot][hv];
        const float dt = x2 - sv.x, ds = sv.y;
        float4 dp = fma4(ds, a1v, acc);
        dp = fma4(dt, a2v, dp);
        st4(A.dP + row * K + cq, dp);
        da1 = fma4(ds, Pj, da1);
        da2 = fma4(dt, Pj, da2);
        acc = accv = f4(0.f);
      }
    };
    const TP* Gl = Gb + cq;
#pragma unroll 1
    for (int g0 = 0; g0 < ne; g0 += 2 * GR) {
#pragma unroll
      for (int u = 0; u < GR; ++u) {
        const int e = g0 + GR + u;
        qb[u] = e < ne ? SL::load(Gl + ga.row(sJ[wib][e]) * K, ga.policy(sJ[wib][e])) : SL::zero();
      }
#pragma unroll
      for (int u = 0; u < GR; ++u)
        if (g0 + u < ne) edge(g0 + u, qa[u]);
#pragma unroll
      for (int u = 0; u < GR; ++u) {
        const int e = g0 + 2 * GR + u;
        qa[u] = e < ne ? SL::load(Gl + ga.row(sJ[wib][e < 32 ? e : 0]) * K,
                                  ga.policy(sJ[wib][e < 32 ? e : 0]))
                       : SL::zero();
      }
#pragma unroll
      for (int u = 0; u < GR; ++u)
        if (g0 + GR + u < ne) edge(g0 + GR + u, qb[u]);
    }
    __syncwarp();
    cur = nxt;
  }
  st4(A.da_part + (da_row0 + gw) * 2 * K + cq, da1);
  st4(A.da_part + (da_row0 + gw) * 2 * K + K + cq, da2);
}

// short rows without stored entries: Z = 0, H_out = sigma(0), Q = 0, m = l = 0
// (forward); dP = 0 (backward: ds = G.Q = 0, no entries)
__global__ void gat_empty_rows_kernel(const int4* __restrict__ meta, int64_t n, GatFwdOut o,
                                      float* __restrict__ dP, int act, int NH) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const float4 hz = act_fwd4(act, f4(0.f));
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < n; w += nw) {
    const int64_t row = __ldg(meta + w).x;
    if (dP) {
      st4(dP + row * K + lane * 4, f4(0.f));
      continue;
    }
    if (o.Z) st4(o.Z + row * K + lane * 4, f4(0.f));
    st4(o.Hout + row * K + lane * 4, hz);
    if (o.Q) st4(o.Q + row * K + lane * 4, f4(0.f));
    if (o.m && lane < NH) {
      o.m[row * NH + lane] = 0.f;
      o.l[row * NH + lane] = 0.f;
    }
  }
}

template <typename F>
int grid_of_fn(F* f) {
  return persistent_blocks(reinterpret_cast<const void*>(f));
}

}  // namespace

#define AGNN_BUNDLE_DISPATCH(NH_, CALL)                                 \
  do {                                                                  \
    if (NH_ == 1) { constexpr int NH = 1; CALL; }                       \
    else if (NH_ == 2) { constexpr int NH = 2; CALL; }                  \
    else if (NH_ == 4) { constexpr int NH = 4; CALL; }                  \
    else if (NH_ == 8) { constexpr int NH = 8; CALL; }                  \
    else return fail(AGNN_EUNSUPPORTED, "GAT k'=128: heads must be 1/2/4/8"); \
  } while (0)

// bundles run for fp32 storage by default (agnn_plan_options.short_bundles; measured
// C5, round 1: fwd short rows 14.0 -> 12.3 ms, bwd 13.3 -> 12.9 ms); for bf16 they
// measured on par or slightly slower than the row-group kernels (10.3 -> 10.8 ms).
// 2 resident 256-thread blocks per SM (3 measured slower: fwd 12.2 -> 15.1 ms).

template <typename TP>
agnn_status gat_fwd_bundle(const Items& it, int heads, const TP* P, const float* st, float slope,
                           int act, const GatFwdOut& o, cudaStream_t s) {
  if (it.n_short > it.n_short_nz) {
    gat_empty_rows_kernel<<<kNumSMs * 4, 256, 0, s>>>(it.short_meta + it.n_short_nz,
                                                     it.n_short - it.n_short_nz, o, nullptr, act,
                                                     heads);
    AGNN_LAUNCH_CHECK("gat_empty_rows_kernel");
  }
  if (it.n_bundles == 0) return AGNN_OK;
  AGNN_BUNDLE_DISPATCH(heads, ({
    auto* kern = o.Q ? gat_fwd_bundle_kernel<TP, NH, true, 2> : gat_fwd_bundle_kernel<TP, NH, false, 2>;
    kern<<<grid_of_fn(kern), 256, 0, s>>>(it, P, st, slope, act, o);
    AGNN_LAUNCH_CHECK("gat_fwd_short_kernel");
  }));
  return AGNN_OK;
}
template agnn_status gat_fwd_bundle<float>(const Items&, int, const float*, const float*, float,
                                           int, const GatFwdOut&, cudaStream_t);
template agnn_status gat_fwd_bundle<bf16>(const Items&, int, const bf16*, const float*, float, int,
                                          const GatFwdOut&, cudaStream_t);

agnn_status gat_bwd_bundle(const Items& it, int heads, const GatBwdArgs& A, int64_t da_row0,
                           int64_t* warps, cudaStream_t s) {
  *warps = 0;
  if (it.n_short > it.n_short_nz) {
    GatFwdOut none{};
    gat_empty_rows_kernel<<<kNumSMs * 4, 256, 0, s>>>(it.short_meta + it.n_short_nz,
                                                     it.n_short - it.n_short_nz, none, A.dP, 0,
                                                     heads);
    AGNN_LAUNCH_CHECK("gat_empty_rows_kernel");
  }
  if (it.n_bundles == 0) return AGNN_OK;
  AGNN_BUNDLE_DISPATCH(heads, ({
    using KB = void (*)(Items, GatBwdArgs, int64_t);
    KB kern = A.P16 ? (KB)gat_bwd_bundle_kernel<bf16, NH, 2> : (KB)gat_bwd_bundle_kernel<float, NH, 2>;
    const int grid = grid_of_fn(kern);
    kern<<<grid, 256, 0, s>>>(it, A, da_row0);
    AGNN_LAUNCH_CHECK("gat_bwd_short_kernel");
    *warps = (int64_t)grid * 8;
  }));
  return AGNN_OK;
}

}  // namespace agnn
