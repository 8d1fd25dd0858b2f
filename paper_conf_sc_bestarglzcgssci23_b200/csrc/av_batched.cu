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
#include "tcgen05.cuh"
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

// The aggregation of one work item (a light row, or a chunk [beg, end) of a heavy
// row) of global row grow: acc = sum_j w_ij H_j over the item's entries with
// w = exp(beta cos(H_i, H_j) - |beta|) (AGNN; l = sum w, warp-reduced, every lane)
// or w = H_i . H_j (VA; l = 0).  Lane q owns columns 4q..4q+3 of every 128-column
// block.
template <int K, int MODEL, int B, typename TP>
__device__ __forceinline__ float av_fwd_item(const Items& it, const AvFwd& A, const Gath& ga,
                                             int64_t grow, int64_t beg, int64_t end, int lane,
                                             float4 (&acc)[K / 128]) {
  constexpr int V = K / 128;
  using TR = Transpose<B>;
  using SL = Slice<TP>;
  const TP* Hrow = pick_row<TP>(A.H, A.H16);
  const int cq = lane * 4;
  const int my_b = TR::edge_of(lane);
  const bool owner = (lane >> TR::T) == 0;
  const float beta = A.beta, bound = A.bound;
  const TP* Hl = Hrow + cq;
  float4 Hi[V];
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
  return l;
}

// X_i = sum_j w_ij H_j (/ l_i for AGNN): every work item of the plan, a warp per item
template <int K, int MODEL, int B, int MINB, typename TP>
__global__ void __launch_bounds__(256, MINB) av_fwd_batched_kernel(Items it, AvFwd A) {
  constexpr int V = K / 128;
  const int lane = threadIdx.x & 31, cq = lane * 4;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const Gath ga(it);  // L2 residency hints of the gathered rows (plan column classes)
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    float4 acc[V];
    const float l = av_fwd_item<K, MODEL, B, TP>(it, A, ga, it.row_begin + row, beg, end, lane, acc);
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

// ---- SpMMM: Z = (Psi H) W fused (Table 2 "SpMMM ... a composition
// of SpMM and MM") ---------------------------------------------------
//
// The whole AGNN / VA forward of a k_in = k_out = 128 layer in one kernel; the
// aggregation rows X_i never go through HBM on their way to the projection.
//
// Every warp of the CTA is a worker that walks the plan's items exactly as
// av_fwd_batched_kernel does (heavy-row chunks first, then light rows, statically
// strided over the grid, B-edge batches).  A light row's X_i is final when its item
// ends; a chunk writes its partial (pacc, pl) and counts itself in its heavy row's
// counter, and the warp that completes the count merges the row's partials in
// ascending chunk order (the arithmetic of av_fwd_merge_kernel, so X is bitwise
// that of the unfused path).  Each finished row, split into tf32 hi/lo, goes to
// the next position of a shared-memory tile of NROW rows (the UMMA B operand,
// K-major SWIZZLE_128B).  The warp that completes a tile issues tcgen05.mma
// kind::tf32 with A = W^T resident in tensor memory (hi and lo, loaded once per
// CTA), so TMEM receives Z^T of the tile (lane = output feature, column = tile
// position): Z = Xh Wh + Xl Wh + Xh Wl (3xTF32, the K loop spread over NG
// accumulators as in gemm_tc.cu).  Between their items, warps read it back (a warp
// reaches the TMEM lane quarter warp % 4: 32 output features; each quarter of a
// tile is claimed by the first free warp of that quarter), apply sigma and store Z
// (training) and H_out by row id.  A ring of S tiles lets the tile being multiplied
// and stored overlap the next ones' rows; the last warp to finish pads the CTA's
// partial last tile.
//
// Per ring slot b (tile t, use u = t / S):
//   producer: take a position (CTA counter), wait epi_done[b] >= u (slot and its TMEM
//             accumulators free; the waiting warp stores finished tiles meanwhile),
//             write the row + its id, fence.proxy.async, count it in tile_cnt[b];
//             the NROW-th issues the MMAs (-> mma_full[b]) after arriving on
//             rows_ready[b] (the row ids, released to the epilogue);
//   quarter q: mma_full[b] done and qnext[q] == t claimed -> tcgen05.ld the 32
//             features, store, count in epi_cnt[b]; the fourth sets epi_done[b] = u + 1.
// (epi_done is a counter, not an mbarrier: a warp held up by a long row may take a
// slot's next use while the ring has moved on by more than one phase.)
struct SpmmmOut {
  const float* W;  // [128 x 128] row-major (k_in x k_out)
  float* Z;        // [n_local x 128] pre-activation (training; nullable)
  float* H_out;    // [n_local x 128] sigma(Z)
  int* hcnt;       // [n_heavy] completed chunks per heavy row (zeroed by the launcher)
  int act;
  int store_x;     // training: X and l are stored too (the backward reads them)
};

constexpr int SP_NROW = 32;  // rows per tile (UMMA N)
constexpr int SP_S = 4;      // ring slots (2: same time, measured)
constexpr int SP_NG = 2;     // accumulation groups (K = 128 in 32-column chunks)
constexpr int SP_SLOT_BYTES = SP_NROW * 128 * 4;  // one of hi / lo

__device__ __forceinline__ bool mbar_test(uint64_t* b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      "selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(s_addr(b)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ float4 ldcg4(const float* p) {
  return __ldcg(reinterpret_cast<const float4*>(p));
}
// heavy row of chunk slot w: the largest h with heavy_off[h] <= w
__device__ __forceinline__ int heavy_of(const Items& it, int64_t w) {
  int lo = 0, hi = (int)it.n_heavy - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (it.heavy_off[mid] <= w) lo = mid;
    else hi = mid - 1;
  }
  return lo;
}

template <int MODEL, int B, typename TP, int NWARP>
__global__ void __launch_bounds__(NWARP * 32, 1)
av_spmmm_kernel(Items it, AvFwd A, SpmmmOut O) {
  constexpr int K = 128, NROW = SP_NROW, S = SP_S, NG = SP_NG;
  static_assert(NWARP >= 4, "warps 0..3 own the TMEM lane quarters");
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NROW >> 3) << 17) |
                             ((uint32_t)(128 >> 4) << 24);
  constexpr uint32_t W_HI = 0, W_LO = 128, D0 = 256;  // TMEM columns
  static_assert(D0 + S * NG * NROW <= 512, "TMEM columns");
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (s_addr(smem_raw) & 1023u)) & 1023u);
  __shared__ uint64_t rows_ready[S], mma_full[S];
  __shared__ int rowid[S][NROW];
  __shared__ int tile_cnt[S], epi_cnt[S], epi_done[S];
  __shared__ int prod, exits, ntiles_final, qnext[4];
  __shared__ uint32_t tmem_base_s;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     s_addr(&tmem_base_s)),
                 "r"(512)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (threadIdx.x < 4) qnext[threadIdx.x] = 0;
  if (threadIdx.x == 0) {
#pragma unroll
    for (int i = 0; i < S; ++i) {
      mbar_init(&rows_ready[i], 1);
      mbar_init(&mma_full[i], 1);
      tile_cnt[i] = epi_cnt[i] = epi_done[i] = 0;
    }
    prod = 0;
    exits = 0;
    ntiles_final = -1;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_s;
  // warp w reaches TMEM lanes 32 (w % 4) .. + 31 = output features m
  const uint32_t lane_base = tmem + ((uint32_t)(32 * (warp & 3)) << 16);
  const int m = 32 * (warp & 3) + lane;
  if (warp < 4) {
    // A = W^T: lane m holds W[k][m], k = 0..127, as tf32 hi (columns 0..127) and lo
    // (columns 128..255)
#pragma unroll 1
    for (int k0 = 0; k0 < K; k0 += 32) {
      float h[32], l[32];
#pragma unroll
      for (int kk = 0; kk < 32; ++kk) split1(__ldg(O.W + (int64_t)(k0 + kk) * 128 + m), h[kk], l[kk]);
      tmem_st32(lane_base + W_HI + (uint32_t)k0, h);
      tmem_st32(lane_base + W_LO + (uint32_t)k0, l);
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();

  volatile int* vdone = epi_done;
  // the MMAs of ring slot b (issued by the thread that completes the tile)
  auto issue = [&](int b) {
    mbar_arrive(&rows_ready[b]);
    tc_fence_after();
    const uint32_t xh = s_addr(smem + b * 2 * SP_SLOT_BYTES), xl = xh + SP_SLOT_BYTES;
#pragma unroll
    for (int kb = 0; kb < K / 32; ++kb) {
      const uint32_t tacc = tmem + D0 + (uint32_t)((b * NG + kb % NG) * NROW);
#pragma unroll
      for (int ks = 0; ks < 4; ++ks) {
        const uint32_t o = (uint32_t)(kb * NROW * 128 + ks * 32);
        const uint32_t acol = (uint32_t)(kb * 32 + ks * 8);
        const uint32_t acc0 = (kb >= NG || ks > 0) ? 1u : 0u;
        mma_tf32_ta(tacc, tmem + W_HI + acol, sw128_desc(xh + o), IDESC, acc0);
        mma_tf32_ta(tacc, tmem + W_HI + acol, sw128_desc(xl + o), IDESC, 1u);
        mma_tf32_ta(tacc, tmem + W_LO + acol, sw128_desc(xh + o), IDESC, 1u);
      }
    }
    mma_commit(&mma_full[b]);
  };
  // store the finished tiles: quarter q = warp % 4 of tile t (TMEM lanes 32q..32q+31,
  // output features 32q..32q+31) can be stored by any of the warps q, q + 4, ..., the
  // first to claim it (qnext[q] = next tile of quarter q), so a warp busy in a long
  // row holds up no tile
  const int qq = warp & 3;
  volatile int* vq = qnext;
  auto service = [&]() {
    for (;;) {
      int t = 0, go = 0;
      if (lane == 0) {
        t = vq[qq];
        const int b = t % S;
        if (mbar_test(&mma_full[b], (uint32_t)((t / S) & 1)) && atomicCAS(&qnext[qq], t, t + 1) == t)
          go = 1;
      }
      if (!__shfl_sync(FULL, go, 0)) return;
      t = __shfl_sync(FULL, t, 0);
      const int b = t % S;
      mbar_wait(&rows_ready[b], (uint32_t)((t / S) & 1));
      tc_fence_after();
      float z[NROW];
#pragma unroll
      for (int gi = 0; gi < NG; ++gi) {
        uint32_t r[NROW];
#pragma unroll
        for (int n0 = 0; n0 < NROW; n0 += 16)
          tmem_ld16_issue(lane_base + D0 + (uint32_t)((b * NG + gi) * NROW + n0), r + n0);
        tmem_ld_wait();
#pragma unroll
        for (int n0 = 0; n0 < NROW; n0 += 16) tmem_reg_fence16(r + n0);
#pragma unroll
        for (int n = 0; n < NROW; ++n) z[n] = gi == 0 ? __uint_as_float(r[n]) : z[n] + __uint_as_float(r[n]);
      }
      tc_fence_before();
#pragma unroll
      for (int n = 0; n < NROW; ++n) {
        const int row = rowid[b][n];
        if (row >= 0) {
          if (O.Z) O.Z[(int64_t)row * 128 + m] = z[n];
          O.H_out[(int64_t)row * 128 + m] = act_fwd(O.act, z[n]);
        }
      }
      __syncwarp();
      if (lane == 0) {
        __threadfence_block();
        if (atomicAdd(&epi_cnt[b], 1) == 3) {
          epi_cnt[b] = 0;
          __threadfence_block();
          vdone[b] = t / S + 1;
        }
      }
    }
  };

  const int cq = lane * 4;
  const Gath ga(it);
  // this lane's 16-byte chunk of a row in the K-major SWIZZLE_128B tile: K block
  // kc = cq / 32 (NROW x 128 B each), chunk cc = (cq % 32) / 4 of the row's 128 B
  const int kc = lane >> 3, cc = lane & 7;
  auto produce = [&](int row, float4 x) {
    int idx = 0;
    if (lane == 0) idx = atomicAdd(&prod, 1);
    idx = __shfl_sync(FULL, idx, 0);
    const int t = idx / NROW, pos = idx % NROW, b = t % S, u = t / S;
    for (;;) {
      int ok = 0;
      if (lane == 0) ok = vdone[b] >= u;
      if (__shfl_sync(FULL, ok, 0)) break;
      service();
      __nanosleep(32);
    }
    __threadfence_block();
    float4 hi, lo;
    split4(x, hi, lo);
    const int off = kc * NROW * 128 + (pos >> 3) * 1024 + (pos & 7) * 128 + ((cc ^ (pos & 7)) << 4);
    uint8_t* slot = smem + b * 2 * SP_SLOT_BYTES;
    *reinterpret_cast<float4*>(slot + off) = hi;
    *reinterpret_cast<float4*>(slot + SP_SLOT_BYTES + off) = lo;
    if (lane == 0) rowid[b][pos] = row;
    fence_proxy_async();
    __syncwarp();
    if (lane == 0) {
      __threadfence_block();
      if (atomicAdd(&tile_cnt[b], 1) == NROW - 1) {
        tile_cnt[b] = 0;
        __threadfence_block();
        issue(b);
      }
    }
    __syncwarp();
  };

  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t nw = (int64_t)gridDim.x * NWARP;
  for (int64_t w = (int64_t)blockIdx.x * NWARP + warp; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    float4 acc[1];
    float l = av_fwd_item<K, MODEL, B, TP>(it, A, ga, it.row_begin + row, beg, end, lane, acc);
    if (slot >= 0) {  // heavy-row chunk: partial, and the merge if it completes the row
      st4(A.pacc + slot * K + cq, acc[0]);
      if (MODEL == AV_AG && lane == 0) A.pl[slot] = l;
      __threadfence();  // every lane's partial is visible before lane 0 counts it
      __syncwarp();
      int h = 0, last = 0;
      if (lane == 0) {
        h = heavy_of(it, slot);
        const int nch = it.heavy_off[h + 1] - it.heavy_off[h];
        last = atomicAdd(O.hcnt + h, 1) == nch - 1;
      }
      last = __shfl_sync(FULL, last, 0);
      if (!last) {
        service();
        continue;
      }
      h = __shfl_sync(FULL, h, 0);
      __threadfence();
      acc[0] = f4(0.f);
      l = 0.f;
      for (int64_t s2 = it.heavy_off[h]; s2 < it.heavy_off[h + 1]; ++s2) {
        acc[0] = add4(acc[0], ldcg4(A.pacc + s2 * K + cq));
        if (MODEL == AV_AG) l += __ldcg(A.pl + s2);
      }
    }
    const float inv = (MODEL == AV_AG) ? (l > 0.f ? 1.f / l : 0.f) : 1.f;
    const float4 x = mul4(inv, acc[0]);
    if (O.store_x) {
      st4(A.X + row * K + cq, x);
      if (MODEL == AV_AG && lane == 0) A.l[row] = l;
    }
    produce((int)row, x);
    service();
  }
  // the last warp out pads the partial last tile (and issues it) and publishes the
  // tile count
  if (lane == 0) {
    __threadfence_block();
    if (atomicAdd(&exits, 1) == NWARP - 1) {
      const int P = atomicAdd(&prod, 0);
      const int nt = (P + NROW - 1) / NROW;
      if (P % NROW) {
        const int b = (nt - 1) % S, u = (nt - 1) / S;
        while (vdone[b] < u) __nanosleep(32);  // (the slot's writers waited for it already)
        __threadfence_block();
        const int pad = NROW - P % NROW;
        for (int pos = P % NROW; pos < NROW; ++pos) rowid[b][pos] = -1;
        __threadfence_block();
        if (atomicAdd(&tile_cnt[b], pad) == NROW - pad) {
          tile_cnt[b] = 0;
          __threadfence_block();
          issue(b);
        }
      }
      __threadfence_block();
      *reinterpret_cast<volatile int*>(&ntiles_final) = nt;
    }
  }
  __syncwarp();
  // every warp helps store the remaining tiles of its quarter
  for (;;) {
    service();
    int done = 0;
    if (lane == 0) {
      const int nt = *reinterpret_cast<volatile int*>(&ntiles_final);
      done = nt >= 0 && vq[qq] >= nt;
    }
    if (__shfl_sync(FULL, done, 0)) break;
    __nanosleep(64);
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512)
                 : "memory");
}

// 16 warps (one CTA per SM, 128 registers) with 8-edge batches, the residency of
// av_fwd_batched_kernel; measured alternatives (C3, ms per 3-layer forward): 12
// workers + 4 dedicated epilogue warps 13.8, 16 + 4 with 4-edge batches 12.1, this
// 12.5, against 9.0 for av_fwd_batched_kernel + merge + GEMM
constexpr int SP_NWARP = 16;
constexpr int SP_B = 8;
constexpr size_t SP_SMEM = (size_t)SP_S * 2 * SP_SLOT_BYTES + 1024;

template <int MODEL, typename TP>
void launch_spmmm(const Items& it, const AvFwd& A, const SpmmmOut& O, cudaStream_t s) {
  auto k = av_spmmm_kernel<MODEL, SP_B, TP, SP_NWARP>;
  static bool attr = false;  // (first call per instantiation; host-side, not a hot path)
  if (!attr) {
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SP_SMEM);
    attr = true;
  }
  k<<<kNumSMs, SP_NWARP * 32, SP_SMEM, s>>>(it, A, O);
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

agnn_status av_fwd_spmmm(const Items& it, bool agnn, const AvFwd& A, const float* W, float* Z,
                         float* H_out, int* hcnt, int act, bool store_x, cudaStream_t s) {
  if (it.n_light + it.n_chunks == 0) return AGNN_OK;
  if (it.n_heavy > 0) AGNN_CUDA_TRY(cudaMemsetAsync(hcnt, 0, sizeof(int) * it.n_heavy, s));
  const SpmmmOut O{W, Z, H_out, hcnt, act, store_x ? 1 : 0};
  if (A.H16) {
    if (agnn) launch_spmmm<AV_AG, bf16>(it, A, O, s);
    else launch_spmmm<AV_VA, bf16>(it, A, O, s);
  } else {
    if (agnn) launch_spmmm<AV_AG, float>(it, A, O, s);
    else launch_spmmm<AV_VA, float>(it, A, O, s);
  }
  AGNN_LAUNCH_CHECK("av_spmmm_kernel");
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
