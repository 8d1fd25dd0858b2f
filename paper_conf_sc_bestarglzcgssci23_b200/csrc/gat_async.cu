// gat_async.cu — GAT k' = 128 backward for BF16 storage (reading B1) with the
// gathers staged through shared memory by cp.async, so the bytes in flight are
// no longer bounded by registers.
//
// Arithmetic: identical to gat_bwd_k128_kernel<bf16> (same batches of B edges, the
// same transposed reduction, the same fixed summation order), so the outputs are
// bitwise the same; PAPER.md:250-254 (Eq. 6 with Psi^T, readings A11/A12), scores
// in log2 units.
//
// Why: the register kernel holds one batch of 8 edges (2 rows x 256 B each) in
// flight per warp while it computes the previous one; with 16 warps per SM that
// is ~64 KB in flight, and at the loaded DRAM latency (~1.8 us) that caps the
// kernel at ~5.2 TB/s (ncu: DRAM 64 %, 0.6 eligible warps per scheduler).  Here
// each warp keeps NS - 1 stages of B edges in flight in its own shared-memory
// ring (LDGSTS, 16-byte pieces: the P and G rows of the stage's edges plus their
// {s, m, 1/l, delta} records and t values); one 8-warp block per SM with
// NS = 4 is ~96 KB of rows in flight per SM.
//
// Pipeline (per warp, per work item = one light row or one heavy-row chunk):
//   producer step t: copy stage t (B edges) using the column ids loaded at step
//   t - 1, then load the ids of stage t + 1 (one LDG per lane, a whole step to
//   land); consumer step s: wait for stage s (cp.async.wait_group NS - 1: every
//   step commits one group, empty ones included), compute it from shared memory.
//   The ring drains at item boundaries (items are >= short_max + 1 edges long).
#include "gat_args.cuh"
#include "warp_batch.cuh"

namespace agnn {
namespace {

using wb::item_of;
using wb::Transpose;

constexpr unsigned FULL = 0xffffffffu;
constexpr int K = 128;

__device__ __forceinline__ uint32_t saddr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
template <int BYTES>
__device__ __forceinline__ void cp_async(uint32_t dst, const void* src) {
  if constexpr (BYTES == 16)
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
  else
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(dst), "l"(src), "n"(BYTES)
                 : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// one stage of B edges: rows of P and G (bf16, 256 B each), records, t values
template <int NH, int B>
struct Stage {
  static constexpr int ROW = K * 2;                        // bytes per bf16 row
  static constexpr int TB = (4 * NH < 16) ? 16 : 4 * NH;   // t bytes per edge (padded)
  static constexpr int P_OFF = 0, G_OFF = B * ROW, R_OFF = 2 * B * ROW,
                       T_OFF = R_OFF + B * NH * 16;
  static constexpr int BYTES = T_OFF + B * TB;
};

template <int NH>
constexpr int async_batch() { return (K / NH / 4) >= 8 ? 8 : K / NH / 4; }

template <int NH, int NS, int MINB>
__global__ void __launch_bounds__(256, MINB)
gat_bwd_async_kernel(Items it, GatBwdArgs A) {
  constexpr int D = K / NH, HL = D / 4, B = async_batch<NH>();
  static_assert(B <= HL && (B & (B - 1)) == 0, "B edges per batch, at most one per head lane");
  using TR = Transpose<B>;
  using ST = Stage<NH, B>;
  extern __shared__ __align__(16) unsigned char smem[];
  const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
  unsigned char* ring = smem + (size_t)wib * NS * ST::BYTES;
  const uint32_t ring_s = saddr(ring);
  const int hv = lane / HL, ql = lane % HL, cq = lane * 4, gbase = lane & ~(HL - 1);
  const int my_b = TR::edge_of(ql);
  const bool owner = (ql >> TR::T) == 0;
  const int pe = lane % B;  // the edge whose column id this lane loads for the producer
  const float slope = A.slope;
  const int64_t nitems = it.n_chunks + it.n_light;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const unsigned char* Pg = reinterpret_cast<const unsigned char*>(A.P16);
  const unsigned char* Gg = reinterpret_cast<const unsigned char*>(A.G16);
  const unsigned char* Rg = reinterpret_cast<const unsigned char*>(A.rec);
  const unsigned char* Sg = reinterpret_cast<const unsigned char*>(A.st);
  float4 da1 = f4(0.f), da2 = f4(0.f);

  for (int64_t w = gw; w < nitems; w += nw) {
    int64_t row, beg, end, slot;
    item_of(it, w, row, beg, end, slot);
    const int64_t grow = it.row_begin + row;
    const float4 Pj = ldg4(A.P16 + grow * K + cq);
    const float4 Gj = ldg4(A.G16 + grow * K + cq);
    const float4 rj = __ldg(A.rec + grow * NH + hv);  // {s_j, m_j, 1/l_j, delta_j}
    const float tj = __ldg(A.st + grow * (2 * NH) + NH + hv);
    const int nst = (int)((end - beg + B - 1) / B);
    // copy stage t into ring slot t % NS; lane e < B holds the id of edge e in pc.
    // Instruction k moves rows 2k, 2k+1 of the stage's 2B rows (P rows of edges
    // 0..B-1, then their G rows): 16 lanes per row, consecutive 16-byte pieces,
    // so both the global reads and the shared-memory writes are contiguous
    // (no bank conflicts).  Then the records (NH pieces per edge) and t.
    auto produce = [&](int t, int pc) {
      if (t < nst) {
        const int64_t e0 = beg + (int64_t)t * B;
        const int cnt = (int)min((int64_t)B, end - e0);
        const uint32_t sb = ring_s + (uint32_t)((t % NS) * ST::BYTES);
        const int half = lane >> 4, piece = lane & 15;
#pragma unroll
        for (int k = 0; k < B; ++k) {
          const int r = 2 * k + half;            // 0 .. 2B-1
          const int e = r < B ? r : r - B;       // edge of the row
          const int64_t i = (int64_t)(uint32_t)__shfl_sync(FULL, pc, e);
          if (e < cnt)
            cp_async<16>(sb + (uint32_t)(r * ST::ROW + piece * 16),
                         (r < B ? Pg : Gg) + i * ST::ROW + piece * 16);
        }
        {
          const int e = lane / NH, r = lane % NH;  // B * NH <= 32 record pieces
          const int64_t i = (int64_t)(uint32_t)__shfl_sync(FULL, pc, e < B ? e : 0);
          if (e < cnt)
            cp_async<16>(sb + (uint32_t)(ST::R_OFF + (e * NH + r) * 16), Rg + (i * NH + r) * 16);
        }
        {
          constexpr int TP16 = (4 * NH + 15) / 16;  // 16-byte pieces of t per edge (>= 1)
          const int e = lane / TP16, q = lane % TP16;
          const int64_t i = (int64_t)(uint32_t)__shfl_sync(FULL, pc, e < B ? e : 0);
          if (e < cnt) {
            const unsigned char* tsrc = Sg + (i * 2 * NH + NH) * 4;
            if constexpr (4 * NH >= 16)
              cp_async<16>(sb + (uint32_t)(ST::T_OFF + e * ST::TB + q * 16), tsrc + q * 16);
            else
              cp_async<4 * NH>(sb + (uint32_t)(ST::T_OFF + e * ST::TB), tsrc);
          }
        }
      }
      cp_commit();  // one group per step, empty or not
    };
    auto col_of = [&](int t) -> int {
      const int64_t e = beg + (int64_t)t * B + pe;
      return (t < nst && e < end) ? (int)((uint32_t)__ldg(it.col + e) & it.col_mask) : 0;
    };
    // prologue: stages 0 .. NS-2 in flight, the ids of stage NS-1 loading
    {
      int pcs[NS - 1];
#pragma unroll
      for (int t = 0; t < NS - 1; ++t) pcs[t] = col_of(t);
#pragma unroll
      for (int t = 0; t < NS - 1; ++t) produce(t, pcs[t]);
    }
    int pc = col_of(NS - 1);
    float4 acc = f4(0.f);
    float dsp = 0.f, dtp = 0.f;
    for (int s = 0; s < nst; ++s) {
      produce(s + NS - 1, pc);
      pc = col_of(s + NS);
      cp_wait<NS - 1>();
      __syncwarp();
      const unsigned char* sb = ring + (s % NS) * ST::BYTES;
      const int cnt = (int)min((int64_t)B, end - beg - (int64_t)s * B);
      uint2 Pi[B], Gi[B];
#pragma unroll
      for (int b = 0; b < B; ++b) {
        if (b < cnt) {
          Pi[b] = *reinterpret_cast<const uint2*>(sb + ST::P_OFF + b * ST::ROW + cq * 2);
          Gi[b] = *reinterpret_cast<const uint2*>(sb + ST::G_OFF + b * ST::ROW + cq * 2);
        } else {
          Pi[b] = Gi[b] = make_uint2(0u, 0u);
        }
      }
      const bool vm = my_b < cnt;
      const float4 ri = vm ? *reinterpret_cast<const float4*>(sb + ST::R_OFF + (my_b * NH + hv) * 16)
                           : f4(0.f);
      const float ti = vm ? *reinterpret_cast<const float*>(sb + ST::T_OFF + my_b * ST::TB + hv * 4)
                          : 0.f;
      float x1[B], x2[B];
#pragma unroll
      for (int b = 0; b < B; ++b) {
        x1[b] = dot4(Gj, bf4_to_f4(Pi[b]));  // G_j . P_i  (row role)
        x2[b] = dot4(bf4_to_f4(Gi[b]), Pj);  // G_i . P_j  (column role)
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
        acc = fma4(ab, bf4_to_f4(Gi[b]), acc);
      }
      __syncwarp();  // every lane is done reading slot s % NS before it is refilled
    }
    cp_wait<0>();  // the empty tail groups
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

}  // namespace

bool gat_bwd_async_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("AGNN_BWD_ASYNC");  // measured slower than the register kernel
    v = (e && e[0] == '1') ? 1 : 0;            // (C5 bf16: 112 vs 97 ms): opt-in
  }
  return v == 1;
}

// BF16 storage only (A.P16 != NULL); items as for gat_bwd_k128 (long rows + chunks)
agnn_status gat_bwd_async(const Items& it, int heads, const GatBwdArgs& A, int64_t* warps,
                          cudaStream_t s) {
  *warps = 0;
  constexpr int NS = 4;
  auto launch = [&](auto* kern, int stage_bytes) -> agnn_status {
    const int smem = 8 * NS * stage_bytes;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return cuda_status(e, "gat_bwd_async: smem attribute");
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, 256, smem);
    int sms = kNumSMs, dev = 0;
    if (cudaGetDevice(&dev) == cudaSuccess)
      cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const int grid = sms * (per_sm > 0 ? per_sm : 1);
    kern<<<grid, 256, smem, s>>>(it, A);
    AGNN_LAUNCH_CHECK("gat_bwd_kernel");
    *warps = (int64_t)grid * 8;
    return AGNN_OK;
  };
  switch (heads) {
    case 1: return launch(gat_bwd_async_kernel<1, NS, 1>, Stage<1, async_batch<1>()>::BYTES);
    case 2: return launch(gat_bwd_async_kernel<2, NS, 1>, Stage<2, async_batch<2>()>::BYTES);
    case 4: return launch(gat_bwd_async_kernel<4, NS, 1>, Stage<4, async_batch<4>()>::BYTES);
    case 8: return launch(gat_bwd_async_kernel<8, NS, 1>, Stage<8, async_batch<8>()>::BYTES);
    default: return fail(AGNN_EUNSUPPORTED, "GAT k'=128: heads must be 1/2/4/8");
  }
}

}  // namespace agnn
