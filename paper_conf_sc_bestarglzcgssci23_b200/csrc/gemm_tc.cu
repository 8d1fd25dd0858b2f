// gemm_tc.cu — tcgen05 (5th-gen tensor core) GEMM for the dense projections
// (PAPER.md:141 H' = HW, a' = Wa; :149 MM; :211 sigma(Psi H W)).
//
//   C[M x N] = A[M x K] * B^T,   A row-major (K-major), B given as [N x K] (K-major)
//
// FP32 accuracy on TF32 tensor cores with the 3xTF32 split (A = Ah + Al,
// B = Bh + Bl, Ah/Bh = fp32 rounded to tf32, Al/Bl = the remainders rounded to
// tf32; C = Ah Bh + Ah Bl + Al Bh accumulated in fp32 TMEM).  The
// projections are HBM-bound (AI = 32 FLOP/B at k = 128 against a TF32 ridge
// of ~170), so the 3 MMAs cost nothing in wall time.
//
// Structure (one CTA of 128 threads per SM, persistent over 128-row tiles):
//   * B (<= 160 x 128 fp32) is split once per CTA into hi/lo tiles in shared
//     memory in the UMMA K-major SWIZZLE_128B layout;
//   * A arrives by TMA (cp.async.bulk.tensor, 128B swizzle) in 32-column chunks
//     through a 2-stage ring; the 128 threads split each chunk in place;
//   * thread 0 issues tcgen05.mma.kind::tf32 (M=128, N, K=8) x 4 k-steps x 3
//     terms per chunk into a TMEM accumulator and commits to an mbarrier;
//   * the epilogue reads TMEM with tcgen05.ld (32 lanes x 16 columns per warp
//     instruction), applies sigma when asked, and stores the row.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <mutex>

#include "internal.cuh"
#include "tcgen05.cuh"

namespace agnn {
namespace {

constexpr int TC_BM = 128;           // rows per tile (UMMA M)
constexpr int TC_KC = 32;            // fp32 columns per 128-byte swizzle atom
constexpr int TC_THREADS = 128;

__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(s_addr(dst)),
      "l"(map), "r"(s_addr(bar)), "r"(c0), "r"(c1)
      : "memory");
}
// L2 prefetch of a TMA box (no shared memory): the ring holds only 1-2 chunks in
// flight, so chunks further ahead are pulled into L2 to hide the DRAM latency
__device__ __forceinline__ void tma_prefetch_2d(const CUtensorMap* map, int c0, int c1) {
  asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global.tile [%0, {%1, %2}];" ::"l"(map),
               "r"(c0), "r"(c1)
               : "memory");
}
#ifndef AGNN_EXP_PF
#define AGNN_EXP_PF 6
#endif
constexpr int TC_PF = AGNN_EXP_PF;  // chunks prefetched ahead into L2


struct TcOut {
  float* C0;    // columns [0, n_split), row stride n_split (nullable)
  float* C1;    // columns [n_split, n_store), row stride n_store - n_split
  float* Cact;  // sigma(C) for columns < n_split (nullable)
  int n_split, n_store, act;
  bf16* C0h;    // EPI_BF16: columns [0, n_split) stored as bfloat16 here instead of C0
  // EPI_PEER (fused GEMM -> needed-rows exchange): row r also goes to peer pi's
  // replicas pC0[pi] / pC1[pi] (same offsets) when bit pi of pmask[r] is set
  int npeer;
  float* pC0[kMaxPeers - 1];
  float* pC1[kMaxPeers - 1];
  const uint8_t* pmask;
};

// epilogue variants (compile time, so the plain fp32 epilogue carries no peer or
// bf16 code)
constexpr int EPI_PLAIN = 0;  // C0 | C1 fp32 (+ sigma copy)
constexpr int EPI_PEER = 1;   // also the peers' replicas of the rows they reference
constexpr int EPI_BF16 = 2;   // C0 columns rounded to bfloat16 into C0h (reading B1)

// 16 consecutive columns c0.. of output row `row` (C0 | C1 split, optional sigma copy).
__device__ __forceinline__ void store_row16_to(const TcOut& out, float* C0, float* C1, float* Ca,
                                               int64_t row, int c0, const float (&v)[16]) {
#pragma unroll
  for (int j = 0; j < 16; j += 4) {
    const int c = c0 + j;
    const float4 q = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
    if (c + 3 < out.n_split && (out.n_split & 3) == 0) {
      if (C0) st4(C0 + row * out.n_split + c, q);
      if (Ca) st4(Ca + row * out.n_split + c, act_fwd4(out.act, q));
    } else if (c < out.n_split) {
#pragma unroll
      for (int x = 0; x < 4; ++x) {
        if (c + x < out.n_split) {
          if (C0) C0[row * out.n_split + c + x] = v[j + x];
          if (Ca) Ca[row * out.n_split + c + x] = act_fwd(out.act, v[j + x]);
        } else if (c + x < out.n_store) {
          C1[row * (out.n_store - out.n_split) + (c + x - out.n_split)] = v[j + x];
        }
      }
    } else if (c < out.n_store) {
      const int w1 = out.n_store - out.n_split;
#pragma unroll
      for (int x = 0; x < 4; ++x)
        if (c + x < out.n_store) C1[row * w1 + (c + x - out.n_split)] = v[j + x];
    }
  }
}
template <int EPI>
__device__ __forceinline__ void store_row16(const TcOut& out, int64_t row, int c0,
                                            const float (&v)[16]) {
  if constexpr (EPI == EPI_BF16) {
#pragma unroll
    for (int x = 0; x < 16; ++x) {
      const int c = c0 + x;
      if (c < out.n_split) out.C0h[row * out.n_split + c] = __float2bfloat16_rn(v[x]);
      else if (c < out.n_store) out.C1[row * (out.n_store - out.n_split) + (c - out.n_split)] = v[x];
    }
    return;
  }
  store_row16_to(out, out.C0, out.C1, out.Cact, row, c0, v);
  if constexpr (EPI == EPI_PEER) {
    const uint32_t m = out.pmask[row];
#pragma unroll 1
    for (int pi = 0; pi < out.npeer; ++pi)
      if ((m >> pi) & 1u) store_row16_to(out, out.pC0[pi], out.pC1[pi], nullptr, row, c0, v);
  }
}

// 32 columns [c0, c0+32) of the warp's 32 rows [row0, row0+32) through a per-warp
// shared-memory transpose, so every store instruction writes 4 full 128-byte rows
// (a thread-per-row store touches 32 lines per instruction, 8x the L2 write requests)
template <int EPI>
__device__ __forceinline__ void store_block32(const TcOut& out, int64_t row0, int64_t M, int c0,
                                              const float (&v)[32], float* stg, int lane) {
  // stg: [32 rows][36 floats] (16-byte aligned rows, 4-float pad against bank conflicts)
#pragma unroll
  for (int j = 0; j < 32; j += 4)
    *reinterpret_cast<float4*>(stg + lane * 36 + j) = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
  __syncwarp();
  const int rr = lane >> 3, cc = (lane & 7) * 4;
#pragma unroll
  for (int k = 0; k < 8; ++k) {
    const int r = 4 * k + rr;
    const int64_t row = row0 + r;
    const float4 q = *reinterpret_cast<const float4*>(stg + r * 36 + cc);
    if (row < M) {
      if constexpr (EPI == EPI_BF16) {
        st4(out.C0h + row * out.n_split + c0 + cc, q);  // 8 lanes x 8 B: a 64-byte run per row
        continue;
      }
      if (out.C0) st4(out.C0 + row * out.n_split + c0 + cc, q);
      if (out.Cact) st4(out.Cact + row * out.n_split + c0 + cc, act_fwd4(out.act, q));
      if constexpr (EPI == EPI_PEER) {  // NVLink stores to the peers that need this row
        const uint32_t m = out.pmask[row];
#pragma unroll 1
        for (int pi = 0; pi < out.npeer; ++pi)
          if ((m >> pi) & 1u) st4(out.pC0[pi] + row * out.n_split + c0 + cc, q);
      }
    }
  }
  __syncwarp();
}

// Warp-specialised CTA (one per SM, persistent over 128-row tiles), 8 warps:
//   warps 0-3 ("math"): thread 0 keeps the TMA ring S - 1 chunks ahead (plus L2
//     prefetches further out); all 128 threads split each landed chunk in place;
//     thread 0 issues the tcgen05.mma chain and commits to the stage's barrier
//     (stage free) and, after a tile's last chunk, to acc_full;
//   warps 4-7 ("epilogue"): wait acc_full, drain the NG TMEM accumulators into
//     registers (summed with round-to-nearest FADDs), release TMEM (acc_empty)
//     and only then write the rows to global memory — the stores of tile t
//     overlap the loads, splits and MMAs of tile t+1.
// SB = false: B (hi/lo) resident in shared memory, split once per CTA;
// SB = true:  B streamed through the ring with A (wide operands, k = 256).
constexpr int TC_WS_THREADS = 256;

__device__ __forceinline__ void math_barrier() {  // the 128 math threads only
  asm volatile("bar.sync 1, 128;" ::: "memory");
}

template <int N, int K, int S, bool SB, int EPI>
__global__ void __launch_bounds__(TC_WS_THREADS, 1)
gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
               const float* __restrict__ B, int n_real, int64_t M, TcOut out) {
  static_assert(N % 16 == 0 && N >= 16 && N <= 256, "UMMA N for M = 128");
  static_assert(K % TC_KC == 0, "K must be a multiple of 32");
  constexpr int KCH = K / TC_KC;                    // 128-byte chunks along K
  constexpr int A_BYTES = TC_BM * 128;              // one of A hi / lo per stage
  constexpr int BC_BYTES = N * 128;                 // one of B hi / lo per chunk
  constexpr int BRES = SB ? 0 : KCH * BC_BYTES;     // resident B (one of hi / lo)
  constexpr int STAGE = SB ? 2 * A_BYTES + 2 * BC_BYTES : A_BYTES;
  // Accumulation groups: the tensor core rounds the fp32 accumulator once per MMA, so
  // the K loop is spread over NG TMEM accumulators (one per 32-wide K chunk where they
  // fit) that the epilogue adds with round-to-nearest FADDs.
  // LOT (resident B): the A lo part goes to TMEM (2 slots of 32 columns) instead of
  // shared memory, so a stage is 16 KB and the ring holds S - 1 chunks in flight
  constexpr bool LOT = !SB;
  constexpr int LO_SLOTS = 2;  // 32-column TMEM slots of A lo (chunk g uses slot g % 2)
  constexpr int LO_COLS = LOT ? 32 * LO_SLOTS : 0;
  constexpr int NG0 = N <= 128 ? 4 : N <= 160 ? 3 : 2;
  constexpr int NGT = (NG0 * N + LO_COLS <= 512) ? NG0 : (NG0 - 1) * N + LO_COLS <= 512 ? NG0 - 1 : 2;
  constexpr int NG = KCH < NGT ? KCH : NGT;
  constexpr uint32_t LO_COL = (uint32_t)(NG * N);  // first TMEM column of the lo slots
  constexpr uint32_t TMEM_NEED = (uint32_t)(NG * N + LO_COLS);
  static_assert(TMEM_NEED <= 512, "TMEM columns");
  constexpr uint32_t TMEM_COLS = TMEM_NEED <= 32 ? 32 : TMEM_NEED <= 64 ? 64 : TMEM_NEED <= 128 ? 128
                                 : TMEM_NEED <= 256 ? 256 : 512;
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) |
                             ((uint32_t)(TC_BM >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-byte aligned by an offset from the __shared__ array, so every access stays
  // in the shared address space (LDS/STS, not generic loads and stores)
  uint8_t* smem = smem_raw + ((1024u - (s_addr(smem_raw) & 1023u)) & 1023u);
  uint8_t* Bh = smem;                  // resident B (SB = false)
  uint8_t* Bl = smem + BRES;
  uint8_t* ring = smem + 2 * BRES;     // S stages
  float* stg = reinterpret_cast<float*>(ring + S * STAGE);  // epilogue transpose, 4 x 32 x 36
  __shared__ uint64_t tma_bar[S], mma_bar[S], acc_full, acc_empty[NG];
  __shared__ uint32_t tmem_base_s;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const bool math = warp < 4;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     s_addr(&tmem_base_s)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (tid == 0) {
#pragma unroll
    for (int i = 0; i < S; ++i) {
      mbar_init(&tma_bar[i], 1);
      mbar_init(&mma_bar[i], 1);
    }
    mbar_init(&acc_full, 1);
#pragma unroll
    for (int i = 0; i < NG; ++i) mbar_init(&acc_empty[i], 128);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
    if (SB) asm volatile("prefetch.tensormap [%0];" ::"l"(&tmB) : "memory");
  }
  if (!SB) {
    // B -> hi/lo tiles in the swizzled K-major layout (rows >= n_real are zero)
    for (int idx = tid; idx < N * (K / 4); idx += TC_WS_THREADS) {
      const int n = idx / (K / 4), c16 = idx % (K / 4), kc = c16 / 8, cc = c16 % 8;
      float4 v = f4(0.f);
      if (n < n_real) v = ldg4(B + (int64_t)n * K + c16 * 4);
      float4 hi, lo;
      split4(v, hi, lo);
      const int off = kc * N * 128 + (n >> 3) * 1024 + (n & 7) * 128 + ((cc ^ (n & 7)) << 4);
      *reinterpret_cast<float4*>(Bh + off) = hi;
      *reinterpret_cast<float4*>(Bl + off) = lo;
    }
    fence_proxy_async();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_s;

  const int64_t ntiles = (M + TC_BM - 1) / TC_BM;
  const int64_t first = blockIdx.x;
  const int64_t my_tiles = first < ntiles ? (ntiles - 1 - first) / gridDim.x + 1 : 0;

  if (math) {
    const int64_t nchunks = my_tiles * KCH;
    auto issue = [&](int64_t g) {
      const int st = (int)(g % S);
      const int64_t t = first + (g / KCH) * gridDim.x;
      const int kcol = (int)(g % KCH) * TC_KC;
      uint8_t* base = ring + st * STAGE;
      mbar_expect_tx(&tma_bar[st], A_BYTES + (SB ? BC_BYTES : 0));
      tma_load_2d(base, &tmA, &tma_bar[st], kcol, (int)(t * TC_BM));
      if (SB) tma_load_2d(base + 2 * A_BYTES, &tmB, &tma_bar[st], kcol, 0);
    };
    if (tid == 0)
      for (int64_t g = 0; g < S - 1 && g < nchunks; ++g) issue(g);
    for (int64_t g = 0; g < nchunks; ++g) {
      const int st = (int)(g % S);
      const uint32_t par = (uint32_t)((g / S) & 1);
      const int kc = (int)(g % KCH);
      const int64_t tl = g / KCH;  // this CTA's tile ordinal
      mbar_wait(&tma_bar[st], par);
      uint8_t* Ahi = ring + st * STAGE;
      uint8_t* Alo = Ahi + A_BYTES;  // SB only
      const uint32_t lo_slot = LO_COL + (uint32_t)((g % LO_SLOTS) * 32);
      if (LOT) {
        // thread r splits row r of the tile: hi in place (swizzled 128-byte row),
        // lo into TMEM lane r.  The slot was last read by chunk g-LO_SLOTS's MMAs.
        if (g >= LO_SLOTS)
          mbar_wait(&mma_bar[(g - LO_SLOTS) % S], (uint32_t)(((g - LO_SLOTS) / S) & 1));
        uint8_t* rowp = Ahi + tid * 128;
        float lo[32];
#ifndef AGNN_EXP_NOSPLIT
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          float4* q = reinterpret_cast<float4*>(rowp + ((c ^ (tid & 7)) << 4));
          float4 hi, l4;
          split4(*q, hi, l4);
          *q = hi;
          lo[4 * c] = l4.x;
          lo[4 * c + 1] = l4.y;
          lo[4 * c + 2] = l4.z;
          lo[4 * c + 3] = l4.w;
        }
        tc_fence_after();
        tmem_st32(tmem + ((uint32_t)(warp * 32) << 16) + lo_slot, lo);
#endif
      } else {
        constexpr int SPLIT16 = (A_BYTES + (SB ? BC_BYTES : 0)) / 16;
#pragma unroll 4
        for (int i = tid; i < SPLIT16; i += 128) {
          const bool isA = !SB || i < A_BYTES / 16;
          uint8_t* hp = isA ? Ahi + i * 16 : Ahi + 2 * A_BYTES + (i - A_BYTES / 16) * 16;
          uint8_t* lp = hp + (isA ? A_BYTES : BC_BYTES);
          float4 hi, lo;
          split4(*reinterpret_cast<const float4*>(hp), hi, lo);
          *reinterpret_cast<float4*>(hp) = hi;
          *reinterpret_cast<float4*>(lp) = lo;
        }
      }
      fence_proxy_async();
      tc_fence_before();
      math_barrier();
      if (tid == 0) {
        const int grp = kc % NG;
        // the first MMA into an accumulator group of a tile overwrites it: the epilogue
        // must have drained that group of the previous tile (groups are released one by
        // one, so the drain overlaps this tile's first chunks)
        if (kc < NG && tl >= 1) mbar_wait(&acc_empty[grp], (uint32_t)((tl - 1) & 1));
        tc_fence_after();
        const uint32_t ah = s_addr(Ahi), al = s_addr(Alo);
        const uint32_t bh = SB ? s_addr(Ahi + 2 * A_BYTES) : s_addr(Bh + kc * BC_BYTES);
        const uint32_t bl = SB ? bh + BC_BYTES : s_addr(Bl + kc * BC_BYTES);
        const uint32_t tacc = tmem + (uint32_t)(grp * N);
#pragma unroll
        for (int ks = 0; ks < TC_KC / 8; ++ks) {  // K = 8 tf32 (32 bytes) per MMA
          const uint32_t o = ks * 32;
          const uint32_t acc0 = (kc >= NG || ks > 0) ? 1u : 0u;  // first MMA of the group
          mma_tf32(tacc, sw128_desc(ah + o), sw128_desc(bh + o), IDESC, acc0);
#ifdef AGNN_EXP_NOSPLIT
          if (LOT) continue;
#endif
          mma_tf32(tacc, sw128_desc(ah + o), sw128_desc(bl + o), IDESC, 1u);
          if (LOT) mma_tf32_ta(tacc, tmem + lo_slot + (uint32_t)(ks * 8), sw128_desc(bh + o), IDESC, 1u);
          else mma_tf32(tacc, sw128_desc(al + o), sw128_desc(bh + o), IDESC, 1u);
        }
        mma_commit(&mma_bar[st]);
        if (kc == KCH - 1) mma_commit(&acc_full);
        // refill the stage of chunk g-1 with chunk g+S-1 once chunk g-1's MMAs are done:
        // waiting here (after chunk g's MMAs are queued behind them) keeps the tensor
        // pipe busy while the math warps split chunk g+1
        if (g + S - 1 + TC_PF < nchunks) {
          const int64_t gp = g + S - 1 + TC_PF;
          tma_prefetch_2d(&tmA, (int)(gp % KCH) * TC_KC,
                          (int)((first + (gp / KCH) * gridDim.x) * TC_BM));
        }
        if (g + S - 1 < nchunks) {
          if (g >= 1) mbar_wait(&mma_bar[(g - 1) % S], (uint32_t)(((g - 1) / S) & 1));
          issue(g + S - 1);
        }
      }
    }
  } else {
    const int ew = warp - 4;  // TMEM lanes 32 ew .. 32 ew + 31
    for (int64_t tl = 0; tl < my_tiles; ++tl) {
      mbar_wait(&acc_full, (uint32_t)(tl & 1));
      tc_fence_after();
      const uint32_t tbase = tmem + ((uint32_t)(ew * 32) << 16);
      const int64_t t = first + tl * gridDim.x;
      const int64_t row0 = t * TC_BM + ew * 32;
      const int64_t row = row0 + lane;
      // wide tiles drain in two halves (registers); the groups are released after the
      // last half reads them
      constexpr int NP = N > 160 ? N / 2 : N;
#pragma unroll 1
      for (int h0 = 0; h0 < N; h0 += NP) {
        float v[NP];
        const bool last_half = h0 + NP >= N;
        // group-major: all of group 0 (one wait), then each further group added with
        // round-to-nearest FADDs; a group is released as soon as it has been read
#pragma unroll
        for (int gi = 0; gi < NG; ++gi) {
          uint32_t r[NP];
#pragma unroll
          for (int c0 = 0; c0 < NP; c0 += 16) tmem_ld16_issue(tbase + (uint32_t)(gi * N) + h0 + c0, r + c0);
          tmem_ld_wait();
#pragma unroll
          for (int c0 = 0; c0 < NP; c0 += 16) tmem_reg_fence16(r + c0);
          if (last_half) {
            tc_fence_before();
            mbar_arrive(&acc_empty[gi]);
          }
#pragma unroll
          for (int x = 0; x < NP; ++x) v[x] = gi == 0 ? __uint_as_float(r[x]) : v[x] + __uint_as_float(r[x]);
        }
        const bool coal = (out.n_split & 3) == 0;
#ifdef AGNN_EXP_NOSTORE
        if (v[0] != 12345.f) continue;
#endif
#pragma unroll
        for (int c0 = 0; c0 < NP; c0 += 32) {
          if (c0 + 32 <= NP && coal && h0 + c0 + 32 <= out.n_split) {
            float q[32];
#pragma unroll
            for (int x = 0; x < 32; ++x) q[x] = v[c0 + x];
            store_block32<EPI>(out, row0, M, h0 + c0, q, stg + ew * 32 * 36, lane);
          } else if (row < M) {
#pragma unroll
            for (int c1 = c0; c1 < c0 + 32 && c1 < NP; c1 += 16) {
              float q[16];
#pragma unroll
              for (int x = 0; x < 16; ++x) q[x] = v[c1 + x];
              store_row16<EPI>(out, row, h0 + c1, q);
            }
          }
        }
      }
    }
  }
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem),
                 "r"(TMEM_COLS)
                 : "memory");
}

// ---------------------------------------------------------------- C = A^T B
// Weight gradients Y = H^T dP / X^T G (PAPER.md:241 Eq. 5, :298 Eq. 13): the
// reduction runs over the n rows, so both operands are MN-major for the MMA
// (D[k1 x n] += A'[k1 x 8 rows] B'[8 rows x n]).  Each CTA reduces a contiguous
// slab of rows: TMA brings TN_ROWS-row chunks of A and B (128B-swizzled, MN-major
// atoms of 8 rows x 32 columns), threads split them 3xTF32, thread 0 issues
// the MMAs; every TN_GROUP chunks the TMEM accumulator is drained into fp32
// registers (one dW row per thread) so the tensor core's per-MMA rounding
// never compounds over more than TN_GROUP * 3 * TN_ROWS / 8 accumulations.
// 16-row chunks (2 x 32 KB ring stages) so that three CTAs fit one SM (registers: the
// 128-column fp32 dW row per thread): three independent TMA -> split -> MMA chains
// per SM overlap each other's latencies.  Measured at M = 2^24, K1 = N = 128: 32-row
// chunks with one CTA / SM 7.36 ms, 16-row chunks with 2 / SM 5.90 ms, with 3 / SM
// 4.84 ms (scratch/time_gemm.py).  Draining every 4 chunks instead of 2 (64 rows,
// 24 MMA accumulations; test_gpu_gemm.py bounds unchanged): C5 dW 5.1 -> 4.75 ms.
constexpr int TN_ROWS = 16;   // input rows per chunk
constexpr int TN_CTAS = 3;    // resident CTAs per SM
constexpr int TN_GROUP = 4;   // chunks per TMEM drain (64 rows: 24 MMA accumulations)
constexpr int64_t kTnMaxSlabs = 2048;  // fp32 partials per call (summed in fp64)

// MN-major tf32 operands use the 128B swizzle with 32-byte atomicity (the only MN-major
// smem layout for 32-bit types): atoms of 4 rows x 128 B; LBO = stride between
// 32-element MN blocks, SBO = stride between 4-row K groups; layout type 1.
__device__ __forceinline__ uint64_t sw128_mn_desc(uint32_t saddr, uint32_t lbo_bytes,
                                                  uint32_t sbo_bytes) {
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)(lbo_bytes >> 4) << 16) |
         ((uint64_t)(sbo_bytes >> 4) << 32) | ((uint64_t)1 << 46) | ((uint64_t)1 << 61);
}

template <int K1, int N>
__global__ void __launch_bounds__(TC_THREADS, TN_CTAS)
gemm_tn_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                  int64_t M, int64_t rows_per_cta, float* __restrict__ part, int nbx) {
  // output block (blockIdx.y) of a wider product: the K1 x N block at (qa K1, qb N) of
  // A^T B — the CTAs of every block of one slab run together, so the A and B column
  // blocks a slab shares come from DRAM once (L2 serves the other blocks)
  const int qa = (int)blockIdx.y / nbx, qb = (int)blockIdx.y % nbx;
  constexpr uint32_t LBO = TN_ROWS * 128;  // 32-column MN blocks (one TMA box each)
  constexpr uint32_t SBO = 512;            // 4-row K groups
  static_assert(K1 == 128, "the MMA M is the K1 = 128 rows of dW");
  static_assert(N % 32 == 0 && N <= 256, "N in 32-column atoms");
  constexpr int A_BYTES = TN_ROWS * K1 * 4;     // one chunk of A (hi); lo follows
  constexpr int B_BYTES = TN_ROWS * N * 4;
  constexpr int STAGE = 2 * A_BYTES + 2 * B_BYTES;
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 15) | (1u << 16) |
                             ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
  constexpr uint32_t TMEM_COLS = N <= 32 ? 32 : N <= 64 ? 64 : N <= 128 ? 128 : 256;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (s_addr(smem_raw) & 1023u)) & 1023u);
  __shared__ uint64_t tma_bar[2], mma_bar[2];
  __shared__ uint32_t tmem_base_s;
  const int tid = threadIdx.x, warp = tid >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     s_addr(&tmem_base_s)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (tid == 0) {
    mbar_init(&tma_bar[0], 1);
    mbar_init(&tma_bar[1], 1);
    mbar_init(&mma_bar[0], 1);
    mbar_init(&mma_bar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_s;
  const int64_t nslabs = (M + rows_per_cta - 1) / rows_per_cta;
  int64_t G0 = 0;  // chunks this CTA processed in earlier slabs: stage = G & 1, parity = (G >> 1) & 1
  for (int64_t slab = blockIdx.x; slab < nslabs; slab += gridDim.x) {
  const int64_t r_beg = slab * rows_per_cta;
  const int64_t r_end = min(M, r_beg + rows_per_cta);
  const int64_t nch = r_end > r_beg ? (r_end - r_beg + TN_ROWS - 1) / TN_ROWS : 0;
  float acc[N];
#pragma unroll
  for (int c = 0; c < N; ++c) acc[c] = 0.f;
  auto issue_tma = [&](int64_t g, int st) {
    uint8_t* base = smem + st * STAGE;
    const int r = (int)(r_beg + g * TN_ROWS);
    mbar_expect_tx(&tma_bar[st], A_BYTES + B_BYTES);
#pragma unroll
    for (int b = 0; b < K1 / 32; ++b)
      tma_load_2d(base + b * (TN_ROWS * 128), &tmA, &tma_bar[st], qa * K1 + b * 32, r);
#pragma unroll
    for (int b = 0; b < N / 32; ++b)
      tma_load_2d(base + 2 * A_BYTES + b * (TN_ROWS * 128), &tmB, &tma_bar[st], qb * N + b * 32, r);
  };
  if (tid == 0 && nch > 0) issue_tma(0, (int)(G0 & 1));
  for (int64_t g = 0; g < nch; ++g) {
    const int64_t G = G0 + g;
    const int st = (int)(G & 1);
    if (tid == 0 && g + 1 + TC_PF / 2 < nch) {
      const int r = (int)(r_beg + (g + 1 + TC_PF / 2) * TN_ROWS);
#pragma unroll
      for (int b = 0; b < K1 / 32; ++b) tma_prefetch_2d(&tmA, qa * K1 + b * 32, r);
#pragma unroll
      for (int b = 0; b < N / 32; ++b) tma_prefetch_2d(&tmB, qb * N + b * 32, r);
    }
    if (tid == 0 && g + 1 < nch) {
      // stage st^1 held chunk G-1 (its MMAs must finish before the TMA overwrites it;
      // the previous slab's last chunk was already waited on by its epilogue)
      if (g >= 1) mbar_wait(&mma_bar[st ^ 1], (uint32_t)(((G - 1) >> 1) & 1));
      issue_tma(g + 1, st ^ 1);
    }
    mbar_wait(&tma_bar[st], (uint32_t)((G >> 1) & 1));
    uint8_t* base = smem + st * STAGE;
    // rows past r_end arrive as zeros (TMA out-of-bounds fill) or belong to the next
    // CTA's slab: zero them before the split
    const int64_t rem = r_end - (r_beg + g * TN_ROWS);
    const int valid_rows = rem < TN_ROWS ? (int)rem : TN_ROWS;
#pragma unroll 4
    for (int i = tid; i < (A_BYTES + B_BYTES) / 16; i += TC_THREADS) {
      const bool isA = i < A_BYTES / 16;
      const int li = isA ? i : i - A_BYTES / 16;
      uint8_t* hp = isA ? base + li * 16 : base + 2 * A_BYTES + li * 16;
      uint8_t* lp = hp + (isA ? A_BYTES : B_BYTES);
      const int row = (li * 16 / 128) % TN_ROWS;   // 128-byte row inside a TN_ROWS-row box
      float4 x = *reinterpret_cast<const float4*>(hp);
      if (row >= valid_rows) x = f4(0.f);
      float4 hi, lo;
      split4(x, hi, lo);
      *reinterpret_cast<float4*>(hp) = hi;
      *reinterpret_cast<float4*>(lp) = lo;
    }
    fence_proxy_async();
    tc_fence_before();
    __syncthreads();
    const bool first_in_group = (g % TN_GROUP) == 0;
    if (tid == 0) {
      tc_fence_after();
      const uint32_t ah = s_addr(base), al = ah + A_BYTES;
      const uint32_t bh = s_addr(base + 2 * A_BYTES), bl = bh + B_BYTES;
#pragma unroll
      for (int ks = 0; ks < TN_ROWS / 8; ++ks) {  // 8 input rows per MMA = two 4-row atoms
        const uint32_t o = ks * 1024;
        const uint32_t acc0 = (!first_in_group || ks > 0) ? 1u : 0u;
        mma_tf32(tmem, sw128_mn_desc(ah + o, LBO, SBO), sw128_mn_desc(bh + o, LBO, SBO), IDESC,
                 acc0);
        mma_tf32(tmem, sw128_mn_desc(ah + o, LBO, SBO), sw128_mn_desc(bl + o, LBO, SBO), IDESC, 1u);
        mma_tf32(tmem, sw128_mn_desc(al + o, LBO, SBO), sw128_mn_desc(bh + o, LBO, SBO), IDESC, 1u);
      }
      mma_commit(&mma_bar[st]);
    }
    if ((g % TN_GROUP) == TN_GROUP - 1 || g == nch - 1) {
      mbar_wait(&mma_bar[st], (uint32_t)((G >> 1) & 1));
      tc_fence_after();
      const uint32_t tbase = tmem + ((uint32_t)(warp * 32) << 16);
#pragma unroll
      for (int c0 = 0; c0 < N; c0 += 16) {
        float v[16];
        tmem_ld16(tbase + c0, v);
#pragma unroll
        for (int x = 0; x < 16; ++x) acc[c0 + x] += v[x];
      }
      tc_fence_before();
      __syncthreads();
    }
  }
  // dW row tid of this (block, slab)'s partial
  float* out = part + ((int64_t)blockIdx.y * nslabs + slab) * K1 * N + (int64_t)tid * N;
#pragma unroll
  for (int c = 0; c < N; c += 4) st4(out + c, make_float4(acc[c], acc[c + 1], acc[c + 2], acc[c + 3]));
  G0 += nch;
  }  // slab
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem),
                 "r"(TMEM_COLS)
                 : "memory");
}

// ---------------------------------------------------------------- C = A B^T, roles
// Resident-B shapes (K <= 128): the same product as gemm_tc_kernel with every role
// in its own warp(s), handing chunks on by mbarriers instead of a CTA barrier, so
// no role waits for another's unrelated latency (the TMA issue no longer waits
// behind the split, the split no longer waits for the MMA issue):
//   warp 8  (producer, one lane): chunk g's TMA once the stage's previous MMAs are
//           done (mma_bar), plus L2 prefetches further ahead;
//   warps 0-3 (split): thread r splits row r of the landed chunk, hi in place, lo
//           into a TMEM slot, then arrives on split_bar;
//   warp 9  (MMA, one lane): the 12 tcgen05.mma of a chunk once it is split, into
//           one of two TMEM accumulators (alternate tiles), commits mma_bar /
//           acc_full;
//   warps 4-7 (epilogue): drain the finished accumulator in 32-column parts and
//           store, then release it (acc_empty) — the other accumulator keeps the
//           tensor pipe busy meanwhile.
// Accumulation groups: the tensor core rounds its fp32 accumulator once per MMA, so
// where TMEM holds them (N <= 96: two buffers x two groups) the K chunks alternate
// between NG = 2 accumulators summed by the epilogue; N = 128 / 144 keep one per
// tile (the per-MMA rounding compounds over the tile's 48 MMAs: ~1e-6 normwise).
constexpr int TCR_THREADS = 320;

template <int N, int K, int S, int EPI>
__global__ void __launch_bounds__(TCR_THREADS, 1)
gemm_tc_roles_kernel(const __grid_constant__ CUtensorMap tmA, const float* __restrict__ B,
                     int n_real, int64_t M, TcOut out) {
  static_assert(N % 16 == 0 && N >= 16 && N <= 256, "UMMA N for M = 128");
  static_assert(K % TC_KC == 0 && K <= 128, "resident B, K <= 128");
  constexpr int KCH = K / TC_KC;
  constexpr int A_BYTES = TC_BM * 128;
  constexpr int BC_BYTES = N * 128;
  constexpr int BRES = KCH * BC_BYTES;
  // lo slots: as many as TMEM holds next to the two accumulators, and fewer than the
  // stages (a slot's reuse waits on mma_bar of chunk g - LO_SLOTS, which must not have
  // been reused by a later chunk yet: mbarrier parity tells only adjacent phases apart)
  constexpr int NG = (KCH >= 2 && 4 * N + 2 * 32 <= 512) ? 2 : 1;
  constexpr int LO_T = (2 * NG * N + 4 * 32 <= 512) ? 4 : 2;
  constexpr int LO_SLOTS = LO_T < S - 1 ? LO_T : S - 1;
  static_assert(LO_SLOTS >= 1, "lo slots");
  constexpr uint32_t LO_COL = (uint32_t)(2 * NG * N);
  constexpr uint32_t TMEM_NEED = (uint32_t)(2 * NG * N + 32 * LO_SLOTS);
  static_assert(TMEM_NEED <= 512, "TMEM columns");
  constexpr uint32_t TMEM_COLS = TMEM_NEED <= 32 ? 32 : TMEM_NEED <= 64 ? 64 : TMEM_NEED <= 128 ? 128
                                 : TMEM_NEED <= 256 ? 256 : 512;
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) |
                             ((uint32_t)(TC_BM >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (s_addr(smem_raw) & 1023u)) & 1023u);
  uint8_t* Bh = smem;
  uint8_t* Bl = smem + BRES;
  uint8_t* ring = smem + 2 * BRES;
  float* stg = reinterpret_cast<float*>(ring + S * A_BYTES);  // epilogue transpose, 4 x 32 x 36
  __shared__ uint64_t tma_bar[S], mma_bar[S], split_bar[S], acc_full[2], acc_empty[2];
  __shared__ uint32_t tmem_base_s;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     s_addr(&tmem_base_s)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (tid == 0) {
#pragma unroll
    for (int i = 0; i < S; ++i) {
      mbar_init(&tma_bar[i], 1);
      mbar_init(&mma_bar[i], 1);
      mbar_init(&split_bar[i], 128);
    }
    mbar_init(&acc_full[0], 1);
    mbar_init(&acc_full[1], 1);
    mbar_init(&acc_empty[0], 128);
    mbar_init(&acc_empty[1], 128);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
  }
  // B -> hi/lo tiles in the swizzled K-major layout (rows >= n_real are zero)
  for (int idx = tid; idx < N * (K / 4); idx += TCR_THREADS) {
    const int n = idx / (K / 4), c16 = idx % (K / 4), kc = c16 / 8, cc = c16 % 8;
    float4 v = f4(0.f);
    if (n < n_real) v = ldg4(B + (int64_t)n * K + c16 * 4);
    float4 hi, lo;
    split4(v, hi, lo);
    const int off = kc * N * 128 + (n >> 3) * 1024 + (n & 7) * 128 + ((cc ^ (n & 7)) << 4);
    *reinterpret_cast<float4*>(Bh + off) = hi;
    *reinterpret_cast<float4*>(Bl + off) = lo;
  }
  fence_proxy_async();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_s;
  const int64_t ntiles = (M + TC_BM - 1) / TC_BM;
  const int64_t first = blockIdx.x;
  const int64_t my_tiles = first < ntiles ? (ntiles - 1 - first) / gridDim.x + 1 : 0;
  const int64_t nchunks = my_tiles * KCH;

  if (warp == 8) {  // ---------------------------------------------------- producer
    if (lane == 0) {
      for (int64_t g = 0; g < nchunks; ++g) {
        const int st = (int)(g % S);
        if (g >= S) mbar_wait(&mma_bar[st], (uint32_t)(((g - S) / S) & 1));
        const int64_t t = first + (g / KCH) * gridDim.x;
        mbar_expect_tx(&tma_bar[st], A_BYTES);
        tma_load_2d(ring + st * A_BYTES, &tmA, &tma_bar[st], (int)(g % KCH) * TC_KC, (int)(t * TC_BM));
        const int64_t gp = g + TC_PF;
        if (gp < nchunks)
          tma_prefetch_2d(&tmA, (int)(gp % KCH) * TC_KC, (int)((first + (gp / KCH) * gridDim.x) * TC_BM));
      }
    }
  } else if (warp == 9) {  // ---------------------------------------------- MMA issue
    if (lane == 0) {
      for (int64_t g = 0; g < nchunks; ++g) {
        const int st = (int)(g % S);
        const int kc = (int)(g % KCH);
        const int64_t tl = g / KCH;
        const int b = (int)(tl & 1);
        mbar_wait(&split_bar[st], (uint32_t)((g / S) & 1));
        if (kc == 0 && tl >= 2) mbar_wait(&acc_empty[b], (uint32_t)(((tl - 2) >> 1) & 1));
        tc_fence_after();
        const uint32_t ah = s_addr(ring + st * A_BYTES);
        const uint32_t bh = s_addr(Bh + kc * BC_BYTES), bl = s_addr(Bl + kc * BC_BYTES);
        const uint32_t tacc = tmem + (uint32_t)((b * NG + kc % NG) * N);
        const uint32_t lo_slot = LO_COL + (uint32_t)((g % LO_SLOTS) * 32);
#pragma unroll
        for (int ks = 0; ks < TC_KC / 8; ++ks) {
          const uint32_t o = ks * 32;
          const uint32_t acc0 = (kc >= NG || ks > 0) ? 1u : 0u;  // first MMA of the group
          mma_tf32(tacc, sw128_desc(ah + o), sw128_desc(bh + o), IDESC, acc0);
          mma_tf32(tacc, sw128_desc(ah + o), sw128_desc(bl + o), IDESC, 1u);
          mma_tf32_ta(tacc, tmem + lo_slot + (uint32_t)(ks * 8), sw128_desc(bh + o), IDESC, 1u);
        }
        mma_commit(&mma_bar[st]);
        if (kc == KCH - 1) mma_commit(&acc_full[b]);
      }
    }
  } else if (warp < 4) {  // ------------------------------------------------- split
    for (int64_t g = 0; g < nchunks; ++g) {
      const int st = (int)(g % S);
      mbar_wait(&tma_bar[st], (uint32_t)((g / S) & 1));
      // the TMEM lo slot was last read by chunk g - LO_SLOTS's MMAs
      if (g >= LO_SLOTS) mbar_wait(&mma_bar[(g - LO_SLOTS) % S], (uint32_t)(((g - LO_SLOTS) / S) & 1));
      uint8_t* rowp = ring + st * A_BYTES + tid * 128;
      float lo[32];
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        float4* q = reinterpret_cast<float4*>(rowp + ((c ^ (tid & 7)) << 4));
        float4 hi, l4;
        split4(*q, hi, l4);
        *q = hi;
        lo[4 * c] = l4.x;
        lo[4 * c + 1] = l4.y;
        lo[4 * c + 2] = l4.z;
        lo[4 * c + 3] = l4.w;
      }
      tc_fence_after();
      tmem_st32(tmem + ((uint32_t)(warp * 32) << 16) + LO_COL + (uint32_t)((g % LO_SLOTS) * 32), lo);
      fence_proxy_async();
      tc_fence_before();
      mbar_arrive(&split_bar[st]);
    }
  } else {  // ------------------------------------------------------------- epilogue
    const int ew = warp - 4;  // TMEM lanes 32 ew .. 32 ew + 31
    float* wstg = stg + ew * 32 * 36;
    for (int64_t tl = 0; tl < my_tiles; ++tl) {
      const int b = (int)(tl & 1);
      mbar_wait(&acc_full[b], (uint32_t)((tl >> 1) & 1));
      tc_fence_after();
      const uint32_t tbase = tmem + ((uint32_t)(ew * 32) << 16) + (uint32_t)(b * NG * N);
      const int64_t t = first + tl * gridDim.x;
      const int64_t row0 = t * TC_BM + ew * 32;
      const int64_t row = row0 + lane;
      const bool coal = (out.n_split & 3) == 0;
#pragma unroll 1
      for (int c0 = 0; c0 < N; c0 += 32) {
        float q[32];
#pragma unroll
        for (int gi = 0; gi < NG; ++gi) {
          uint32_t r[32];
          tmem_ld16_issue(tbase + (uint32_t)(gi * N) + c0, r);
          if (c0 + 16 < N) tmem_ld16_issue(tbase + (uint32_t)(gi * N) + c0 + 16, r + 16);
          tmem_ld_wait();
          tmem_reg_fence16(r);
          if (c0 + 16 < N) tmem_reg_fence16(r + 16);
#pragma unroll
          for (int x = 0; x < 32; ++x) q[x] = gi == 0 ? __uint_as_float(r[x]) : q[x] + __uint_as_float(r[x]);
        }
        if (c0 + 32 <= N && coal && c0 + 32 <= out.n_split) {
          store_block32<EPI>(out, row0, M, c0, q, wstg, lane);
        } else if (row < M) {
          float q16[16];
#pragma unroll
          for (int x = 0; x < 16; ++x) q16[x] = q[x];
          store_row16<EPI>(out, row, c0, q16);
          if (c0 + 16 < N) {
#pragma unroll
            for (int x = 0; x < 16; ++x) q16[x] = q[16 + x];
            store_row16<EPI>(out, row, c0 + 16, q16);
          }
        }
      }
      tc_fence_before();
      mbar_arrive(&acc_empty[b]);
    }
  }
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem),
                 "r"(TMEM_COLS)
                 : "memory");
}

// Streamed-B shapes (k = 256: B does not fit next to the ring): the same roles as
// gemm_tc_roles_kernel, with the B chunk travelling with the A chunk through the
// ring (both split by the split warps, lo parts in shared memory) and two TMEM
// accumulators of N columns (2 N <= 512).
template <int N, int K, int S, int EPI>
__global__ void __launch_bounds__(TCR_THREADS, 1)
gemm_tc_roles_sb_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                        int64_t M, TcOut out) {
  static_assert(N % 16 == 0 && N >= 16 && N <= 256, "UMMA N for M = 128");
  static_assert(K % TC_KC == 0, "K in 32-column chunks");
  constexpr int KCH = K / TC_KC;
  constexpr int A_BYTES = TC_BM * 128;
  constexpr int BC_BYTES = N * 128;
  constexpr int STAGE = 2 * A_BYTES + 2 * BC_BYTES;  // A hi | A lo | B hi | B lo
  // K-chunk accumulation groups where two buffers of them fit TMEM (N <= 128):
  // ~1e-6 normwise at K = 256; N = 256 keeps one accumulator (~2e-6, the level of
  // an fp32 dot of length 256)
  constexpr int NG = (4 * N <= 512) ? 2 : 1;
  constexpr uint32_t TMEM_NEED = (uint32_t)(2 * NG * N);
  constexpr uint32_t TMEM_COLS = TMEM_NEED <= 32 ? 32 : TMEM_NEED <= 64 ? 64 : TMEM_NEED <= 128 ? 128
                                 : TMEM_NEED <= 256 ? 256 : 512;
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) |
                             ((uint32_t)(TC_BM >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (s_addr(smem_raw) & 1023u)) & 1023u);
  uint8_t* ring = smem;
  float* stg = reinterpret_cast<float*>(ring + S * STAGE);
  __shared__ uint64_t tma_bar[S], mma_bar[S], split_bar[S], acc_full[2], acc_empty[2];
  __shared__ uint32_t tmem_base_s;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     s_addr(&tmem_base_s)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (tid == 0) {
#pragma unroll
    for (int i = 0; i < S; ++i) {
      mbar_init(&tma_bar[i], 1);
      mbar_init(&mma_bar[i], 1);
      mbar_init(&split_bar[i], 128);
    }
    mbar_init(&acc_full[0], 1);
    mbar_init(&acc_full[1], 1);
    mbar_init(&acc_empty[0], 128);
    mbar_init(&acc_empty[1], 128);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmB) : "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_s;
  const int64_t ntiles = (M + TC_BM - 1) / TC_BM;
  const int64_t first = blockIdx.x;
  const int64_t my_tiles = first < ntiles ? (ntiles - 1 - first) / gridDim.x + 1 : 0;
  const int64_t nchunks = my_tiles * KCH;

  if (warp == 8) {  // ---------------------------------------------------- producer
    if (lane == 0) {
      for (int64_t g = 0; g < nchunks; ++g) {
        const int st = (int)(g % S);
        if (g >= S) mbar_wait(&mma_bar[st], (uint32_t)(((g - S) / S) & 1));
        const int64_t t = first + (g / KCH) * gridDim.x;
        const int kcol = (int)(g % KCH) * TC_KC;
        uint8_t* base = ring + st * STAGE;
        mbar_expect_tx(&tma_bar[st], A_BYTES + BC_BYTES);
        tma_load_2d(base, &tmA, &tma_bar[st], kcol, (int)(t * TC_BM));
        tma_load_2d(base + 2 * A_BYTES, &tmB, &tma_bar[st], kcol, 0);
        const int64_t gp = g + TC_PF;
        if (gp < nchunks)
          tma_prefetch_2d(&tmA, (int)(gp % KCH) * TC_KC, (int)((first + (gp / KCH) * gridDim.x) * TC_BM));
      }
    }
  } else if (warp == 9) {  // ---------------------------------------------- MMA issue
    if (lane == 0) {
      for (int64_t g = 0; g < nchunks; ++g) {
        const int st = (int)(g % S);
        const int kc = (int)(g % KCH);
        const int64_t tl = g / KCH;
        const int b = (int)(tl & 1);
        mbar_wait(&split_bar[st], (uint32_t)((g / S) & 1));
        if (kc == 0 && tl >= 2) mbar_wait(&acc_empty[b], (uint32_t)(((tl - 2) >> 1) & 1));
        tc_fence_after();
        uint8_t* base = ring + st * STAGE;
        const uint32_t ah = s_addr(base), al = ah + A_BYTES;
        const uint32_t bh = s_addr(base + 2 * A_BYTES), bl = bh + BC_BYTES;
        const uint32_t tacc = tmem + (uint32_t)((b * NG + kc % NG) * N);
#pragma unroll
        for (int ks = 0; ks < TC_KC / 8; ++ks) {
          const uint32_t o = ks * 32;
          const uint32_t acc0 = (kc >= NG || ks > 0) ? 1u : 0u;
          mma_tf32(tacc, sw128_desc(ah + o), sw128_desc(bh + o), IDESC, acc0);
          mma_tf32(tacc, sw128_desc(ah + o), sw128_desc(bl + o), IDESC, 1u);
          mma_tf32(tacc, sw128_desc(al + o), sw128_desc(bh + o), IDESC, 1u);
        }
        mma_commit(&mma_bar[st]);
        if (kc == KCH - 1) mma_commit(&acc_full[b]);
      }
    }
  } else if (warp < 4) {  // ------------------------------------------------- split
    for (int64_t g = 0; g < nchunks; ++g) {
      const int st = (int)(g % S);
      mbar_wait(&tma_bar[st], (uint32_t)((g / S) & 1));
      uint8_t* base = ring + st * STAGE;
      // A row tid, then B rows tid, tid + 128 (< N): hi in place, lo at +A_BYTES / +BC_BYTES
      // (the 128-byte swizzle is a permutation inside each row: lo keeps hi's position)
#pragma unroll
      for (int part = 0; part < 1 + (N + 127) / 128; ++part) {
        const int r = part == 0 ? tid : tid + (part - 1) * 128;
        if (part > 0 && r >= N) continue;
        uint8_t* rowp = part == 0 ? base + tid * 128 : base + 2 * A_BYTES + r * 128;
        const int lo_off = part == 0 ? A_BYTES : BC_BYTES;
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const int cs = (c ^ (r & 7)) << 4;  // the swizzled order: conflict-free phases
          float4* q = reinterpret_cast<float4*>(rowp + cs);
          float4 hi, lo;
          split4(*q, hi, lo);
          *q = hi;
          *reinterpret_cast<float4*>(rowp + lo_off + cs) = lo;
        }
      }
      fence_proxy_async();
      tc_fence_before();
      mbar_arrive(&split_bar[st]);
    }
  } else {  // ------------------------------------------------------------- epilogue
    const int ew = warp - 4;
    float* wstg = stg + ew * 32 * 36;
    for (int64_t tl = 0; tl < my_tiles; ++tl) {
      const int b = (int)(tl & 1);
      mbar_wait(&acc_full[b], (uint32_t)((tl >> 1) & 1));
      tc_fence_after();
      const uint32_t tbase = tmem + ((uint32_t)(ew * 32) << 16) + (uint32_t)(b * NG * N);
      const int64_t t = first + tl * gridDim.x;
      const int64_t row0 = t * TC_BM + ew * 32;
      const int64_t row = row0 + lane;
      const bool coal = (out.n_split & 3) == 0;
#pragma unroll 1
      for (int c0 = 0; c0 < N; c0 += 32) {
        float q[32];
#pragma unroll
        for (int gi = 0; gi < NG; ++gi) {
          uint32_t r[32];
          tmem_ld16_issue(tbase + (uint32_t)(gi * N) + c0, r);
          if (c0 + 16 < N) tmem_ld16_issue(tbase + (uint32_t)(gi * N) + c0 + 16, r + 16);
          tmem_ld_wait();
          tmem_reg_fence16(r);
          if (c0 + 16 < N) tmem_reg_fence16(r + 16);
#pragma unroll
          for (int x = 0; x < 32; ++x) q[x] = gi == 0 ? __uint_as_float(r[x]) : q[x] + __uint_as_float(r[x]);
        }
        if (c0 + 32 <= N && coal && c0 + 32 <= out.n_split) {
          store_block32<EPI>(out, row0, M, c0, q, wstg, lane);
        } else if (row < M) {
          float q16[16];
#pragma unroll
          for (int x = 0; x < 16; ++x) q16[x] = q[x];
          store_row16<EPI>(out, row, c0, q16);
          if (c0 + 16 < N) {
#pragma unroll
            for (int x = 0; x < 16; ++x) q16[x] = q[16 + x];
            store_row16<EPI>(out, row, c0 + 16, q16);
          }
        }
      }
      tc_fence_before();
      mbar_arrive(&acc_empty[b]);
    }
  }
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem),
                 "r"(TMEM_COLS)
                 : "memory");
}

PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

template <int N, int K, int S, bool SB>
agnn_status launch_tc(const float* A, int64_t M, const float* B, int n_real, const TcOut& o,
                      cudaStream_t s) {
  auto enc = encode_fn();
  if (!enc) return fail(AGNN_ECUDA, "gemm_tc: cuTensorMapEncodeTiled unavailable");
  CUtensorMap ma, mb;
  cuuint64_t da[2] = {(cuuint64_t)K, (cuuint64_t)M};
  cuuint64_t db[2] = {(cuuint64_t)K, (cuuint64_t)n_real};
  cuuint64_t strides[1] = {(cuuint64_t)K * 4};
  cuuint32_t boxa[2] = {(cuuint32_t)TC_KC, (cuuint32_t)TC_BM};
  cuuint32_t boxb[2] = {(cuuint32_t)TC_KC, (cuuint32_t)N};  // rows >= n_real arrive as zeros
  cuuint32_t es[2] = {1, 1};
  if (enc(&ma, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(A), da, strides, boxa, es,
          CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
          CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return fail(AGNN_ECUDA, "gemm_tc: tensor map encode failed");
  if (SB && enc(&mb, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(B), db, strides, boxb,
                es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return fail(AGNN_ECUDA, "gemm_tc: tensor map encode failed");
  if constexpr (!SB) {
    // resident B: the role-split kernel, as many 16 KB stages as fit next to B
    constexpr int bres = 2 * (K / TC_KC) * N * 128;
    constexpr int SR0 = (232448 - 2048 - bres - 4 * 32 * 36 * 4) / (TC_BM * 128);
    constexpr int SR = SR0 > 8 ? 8 : SR0;
    static_assert(SR >= 2, "ring stages");
    constexpr int smem_r = bres + SR * TC_BM * 128 + 4 * 32 * 36 * 4 + 1024;
    static bool attr_r = false;
    if (!attr_r) {
      cudaFuncSetAttribute(gemm_tc_roles_kernel<N, K, SR, EPI_PLAIN>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, smem_r);
      cudaFuncSetAttribute(gemm_tc_roles_kernel<N, K, SR, EPI_BF16>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, smem_r);
      cudaFuncSetAttribute(gemm_tc_roles_kernel<N, K, SR, EPI_PEER>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, smem_r);
      attr_r = true;
    }
    int sms_r = kNumSMs, dev_r = 0;
    if (cudaGetDevice(&dev_r) == cudaSuccess)
      cudaDeviceGetAttribute(&sms_r, cudaDevAttrMultiProcessorCount, dev_r);
    const int grid_r = (int)std::min<int64_t>((M + TC_BM - 1) / TC_BM, sms_r);
    if (o.C0h)
      gemm_tc_roles_kernel<N, K, SR, EPI_BF16><<<grid_r, TCR_THREADS, smem_r, s>>>(ma, B, n_real, M, o);
    else if (o.npeer > 0)
      gemm_tc_roles_kernel<N, K, SR, EPI_PEER><<<grid_r, TCR_THREADS, smem_r, s>>>(ma, B, n_real, M, o);
    else
      gemm_tc_roles_kernel<N, K, SR, EPI_PLAIN><<<grid_r, TCR_THREADS, smem_r, s>>>(ma, B, n_real, M, o);
    AGNN_LAUNCH_CHECK("gemm_tc_kernel");
    return AGNN_OK;
  }
  if constexpr (SB) {
    constexpr int stage = 2 * TC_BM * 128 + 2 * N * 128;
    constexpr int SR0 = (232448 - 2048 - 4 * 32 * 36 * 4) / stage;
    constexpr int SR = SR0 > 6 ? 6 : SR0;
    static_assert(SR >= 2, "ring stages");
    constexpr int smem_r = SR * stage + 4 * 32 * 36 * 4 + 1024;
    static bool attr_sb = false;
    if (!attr_sb) {
      cudaFuncSetAttribute(gemm_tc_roles_sb_kernel<N, K, SR, EPI_PLAIN>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, smem_r);
      cudaFuncSetAttribute(gemm_tc_roles_sb_kernel<N, K, SR, EPI_BF16>,
                           cudaFuncAttributeMaxDynamicSharedMemorySize, smem_r);
      attr_sb = true;
    }
    int sms_r = kNumSMs, dev_r = 0;
    if (cudaGetDevice(&dev_r) == cudaSuccess)
      cudaDeviceGetAttribute(&sms_r, cudaDevAttrMultiProcessorCount, dev_r);
    const int grid_r = (int)std::min<int64_t>((M + TC_BM - 1) / TC_BM, sms_r);
    if (o.C0h)
      gemm_tc_roles_sb_kernel<N, K, SR, EPI_BF16><<<grid_r, TCR_THREADS, smem_r, s>>>(ma, mb, M, o);
    else
      gemm_tc_roles_sb_kernel<N, K, SR, EPI_PLAIN><<<grid_r, TCR_THREADS, smem_r, s>>>(ma, mb, M, o);
    AGNN_LAUNCH_CHECK("gemm_tc_kernel");
    return AGNN_OK;
  }
  constexpr int smem = (SB ? 0 : 2 * (K / TC_KC) * N * 128) +
                       S * (SB ? 2 * TC_BM * 128 + 2 * N * 128 : TC_BM * 128) + 4 * 32 * 36 * 4 +
                       1024;
  static_assert(smem <= 232448 - 1024, "shared memory");
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(gemm_tc_kernel<N, K, S, SB, EPI_PLAIN>,
                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(gemm_tc_kernel<N, K, S, SB, EPI_BF16>,
                         cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  int sms = kNumSMs, dev = 0;
  if (cudaGetDevice(&dev) == cudaSuccess)
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t ntiles = (M + TC_BM - 1) / TC_BM;
  const int grid = (int)std::min<int64_t>(ntiles, sms);
  if (o.C0h)
    gemm_tc_kernel<N, K, S, SB, EPI_BF16><<<grid, TC_WS_THREADS, smem, s>>>(ma, mb, B, n_real, M, o);
  else
    gemm_tc_kernel<N, K, S, SB, EPI_PLAIN><<<grid, TC_WS_THREADS, smem, s>>>(ma, mb, B, n_real, M, o);
  AGNN_LAUNCH_CHECK("gemm_tc_kernel");
  return AGNN_OK;
}

bool map_rows_box32(CUtensorMap* map, const float* base, int64_t rows, int cols, int ld) {
  auto enc = encode_fn();
  if (!enc) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
  cuuint32_t box[2] = {32, (cuuint32_t)TN_ROWS};
  cuuint32_t es[2] = {1, 1};
  return enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box,
             es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B,
             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// C block q (blockIdx.y; at rows (q / nbx) K1, columns (q % nbx) N; row stride ldc) =
// sum over the slab partials of part[q][p][r][c] (r < K1, c < N)
__global__ void tn_sum_kernel(const float* __restrict__ part, int splits, int K1, int N,
                              float* __restrict__ C, int ldc, int nbx) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t count = (int64_t)K1 * N;
  if (i >= count) return;
  const int q = (int)blockIdx.y;
  const float* pq = part + (int64_t)q * splits * count;
  double s = 0.0;  // fixed order, fp64 across the slab partials
  for (int p = 0; p < splits; ++p) s += (double)pq[(int64_t)p * count + i];
  C[((int64_t)(q / nbx) * K1 + i / N) * ldc + (q % nbx) * N + (i % N)] = (float)s;
}

// C block [K1 x N] (row stride ldc) = A^T B over M rows; A, B column blocks of row
// strides lda, ldb
// C [nby K1 x nbx N] = A^T B over M rows in K1 x N blocks, one launch: A [M x nby K1],
// B [M x nbx N] (row strides = their widths)
template <int K1, int N>
agnn_status launch_tn_tc(const float* A, int nby, int64_t M, const float* B, int nbx, float* C,
                         float* ws, cudaStream_t s) {
  CUtensorMap ma, mb;
  if (!map_rows_box32(&ma, A, M, nby * K1, nby * K1) || !map_rows_box32(&mb, B, M, nbx * N, nbx * N))
    return fail(AGNN_ECUDA, "gemm_tn_tc: tensor map encode failed");
  constexpr int smem = 2 * (2 * TN_ROWS * K1 * 4 + 2 * TN_ROWS * N * 4) + 1024;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(gemm_tn_tc_kernel<K1, N>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         smem);
    attr = true;
  }
  int sms = kNumSMs, dev = 0;
  if (cudaGetDevice(&dev) == cudaSuccess)
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // slabs of >= 8192 rows, at most kTnMaxSlabs of them; each (block, slab) leaves one
  // fp32 partial
  int64_t rps = (M + kTnMaxSlabs - 1) / kTnMaxSlabs;
  rps = std::max<int64_t>(rps, 8192);
  rps = (rps + TN_ROWS - 1) / TN_ROWS * TN_ROWS;
  const int64_t nslabs = (M + rps - 1) / rps;
  const int nblk = nby * nbx;
  const int gx = (int)std::min<int64_t>(nslabs, std::max<int64_t>(1, (int64_t)sms * TN_CTAS / nblk));
  gemm_tn_tc_kernel<K1, N><<<dim3(gx, nblk), TC_THREADS, smem, s>>>(ma, mb, M, rps, ws, nbx);
  AGNN_LAUNCH_CHECK("gemm_tn_kernel");
  const int64_t cnt = (int64_t)K1 * N;
  tn_sum_kernel<<<dim3((unsigned)((cnt + 255) / 256), nblk), 256, 0, s>>>(ws, (int)nslabs, K1, N, C,
                                                                          nbx * N, nbx);
  AGNN_LAUNCH_CHECK("sum_splits_kernel");
  return AGNN_OK;
}

}  // namespace

// C[K1 x N] = A^T B over M rows on tensor cores (K1 = 128 with N in {64, 128}; K1 = 256
// with N in {128, 256} as 128 x 128 blocks); ws holds the slab partials of one block.
// AGNN_EUNSUPPORTED for other shapes.
agnn_status gemm_tn_tc(const float* A, int64_t M, int K1, const float* B, int N, float* C,
                       float* ws, cudaStream_t s) {
  if (M <= 0) return AGNN_EUNSUPPORTED;
  if ((reinterpret_cast<uintptr_t>(A) & 15) || (reinterpret_cast<uintptr_t>(B) & 15))
    return AGNN_EUNSUPPORTED;
  if (K1 == 128 && N == 128) return launch_tn_tc<128, 128>(A, 1, M, B, 1, C, ws, s);
  if (K1 == 128 && N == 64) return launch_tn_tc<128, 64>(A, 1, M, B, 1, C, ws, s);
  // K1 = 256: 128 x 128 blocks of C in one launch
  if (K1 == 256 && (N == 256 || N == 128)) return launch_tn_tc<128, 128>(A, 2, M, B, N / 128, C, ws, s);
  return AGNN_EUNSUPPORTED;
}

// C = A * B^T with B [n_real x K] K-major; columns padded to N_pad (multiple of 16).
// Returns AGNN_EUNSUPPORTED when the shape has no tcgen05 instantiation.
agnn_status gemm_tc(const float* A, int64_t M, int K, const float* B, int n_real, float* C0,
                    int n_split, float* C1, int n_store, float* Cact, int act, cudaStream_t s,
                    bf16* C0h, const PeerOut* peers) {
  if ((reinterpret_cast<uintptr_t>(A) & 15) || (K % 32)) return AGNN_EUNSUPPORTED;
  if (C0h && (Cact || (n_split & 3))) return AGNN_EUNSUPPORTED;
  // the peer epilogue exists for the resident-B (K <= 128) kernel; the shape decides,
  // so every rank agrees on whether the exchange was fused
  if (peers && (K > 128 || C0h || !C0 || peers->n > kMaxPeers - 1)) return AGNN_EUNSUPPORTED;
  const int npad = (n_real + 15) / 16 * 16;
  const bool shape_ok = (K == 128 && (npad == 128 || npad == 144 || npad == 160 || npad == 64)) ||
                        (K == 64 && (npad == 64 || npad == 80 || npad == 128)) ||
                        (K == 256 && (npad == 256 || npad == 128));
  if (!shape_ok) return AGNN_EUNSUPPORTED;
  if (M <= 0) return AGNN_OK;
  TcOut o{C0, C1, Cact, n_split, n_store, act, C0h, 0, {}, {}, nullptr};
  if (peers) {
    o.npeer = peers->n;
    o.pmask = peers->mask;
    for (int i = 0; i < peers->n; ++i) {
      o.pC0[i] = peers->C0[i];
      o.pC1[i] = peers->C1[i];
    }
  }
  // resident B: S = the 16 KB stages that fit next to B (2 x K x N x 4 bytes), <= 8
  if (K == 128 && npad == 128) return launch_tc<128, 128, 4, false>(A, M, B, n_real, o, s);
  if (K == 128 && npad == 144) return launch_tc<144, 128, 3, false>(A, M, B, n_real, o, s);
  if (K == 128 && npad == 160) return launch_tc<160, 128, 2, false>(A, M, B, n_real, o, s);
  if (K == 128 && npad == 64) return launch_tc<64, 128, 8, false>(A, M, B, n_real, o, s);
  if (K == 64 && npad == 64) return launch_tc<64, 64, 8, false>(A, M, B, n_real, o, s);
  if (K == 64 && npad == 80) return launch_tc<80, 64, 8, false>(A, M, B, n_real, o, s);
  if (K == 64 && npad == 128) return launch_tc<128, 64, 8, false>(A, M, B, n_real, o, s);
  if (K == 256 && npad == 256) return launch_tc<256, 256, 2, true>(A, M, B, n_real, o, s);
  if (K == 256 && npad == 128) return launch_tc<128, 256, 3, true>(A, M, B, n_real, o, s);
  return AGNN_EUNSUPPORTED;
}

}  // namespace agnn
