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

namespace agnn {
namespace {

constexpr int TC_BM = 128;           // rows per tile (UMMA M)
constexpr int TC_KC = 32;            // fp32 columns per 128-byte swizzle atom
constexpr int TC_THREADS = 128;

__device__ __forceinline__ uint32_t s_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(s_addr(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(s_addr(b)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred p;\nWAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n}\n" ::"r"(s_addr(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(s_addr(dst)),
      "l"(map), "r"(s_addr(bar)), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
// UMMA shared-memory descriptor: K-major, SWIZZLE_128B, 8-row groups 1024 B apart
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
  return (uint64_t)((saddr & 0x3FFFF) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void mma_tf32(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc,
                                         uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   s_addr(bar))
               : "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float (&v)[16]) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,"
      "%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}
// tf32 split with round-to-nearest (cvt.rna): hi = tf32(x), lo = tf32(x - hi).
// |x - hi - lo| <= 2^-22 |x| and the rounding errors are unbiased, so the
// 3-term product matches an fp32 FFMA dot (truncating splits are biased and
// lose ~2^-21 per element, which the ill-conditioned da1 = P^T ds amplifies).
__device__ __forceinline__ float tf32_rna(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return __uint_as_float(r);
}
__device__ __forceinline__ void split4(float4 x, float4& hi, float4& lo) {
  hi = make_float4(tf32_rna(x.x), tf32_rna(x.y), tf32_rna(x.z), tf32_rna(x.w));
  lo = make_float4(tf32_rna(x.x - hi.x), tf32_rna(x.y - hi.y), tf32_rna(x.z - hi.z),
                   tf32_rna(x.w - hi.w));
}

struct TcOut {
  float* C0;    // columns [0, n_split), row stride n_split (nullable)
  float* C1;    // columns [n_split, n_store), row stride n_store - n_split
  float* Cact;  // sigma(C) for columns < n_split (nullable)
  int n_split, n_store, act;
};

template <int N, int K>
__global__ void __launch_bounds__(TC_THREADS, 1)
gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const float* __restrict__ B, int n_real,
               int64_t M, TcOut out) {
  static_assert(N % 16 == 0 && N >= 16 && N <= 256, "UMMA N for M = 128");
  static_assert(K % TC_KC == 0, "K must be a multiple of 32");
  constexpr int KCH = K / TC_KC;                    // 128-byte chunks along K
  constexpr int B_BYTES = KCH * N * 128;            // one of hi / lo
  constexpr int A_STAGE = TC_BM * 128;              // 16 KB raw / hi
  // Accumulation groups: the tensor core rounds the fp32 accumulator once per MMA
  // (biased), so the K loop is spread over NG TMEM accumulators (one per 32-wide
  // K chunk where they fit) that the epilogue adds with round-to-nearest FADDs.
  constexpr int NG = (KCH < (N <= 128 ? 4 : N <= 160 ? 3 : 2)) ? KCH : (N <= 128 ? 4 : N <= 160 ? 3 : 2);
  constexpr uint32_t TMEM_NEED = (uint32_t)(NG * N);
  constexpr uint32_t TMEM_COLS = TMEM_NEED <= 32 ? 32 : TMEM_NEED <= 64 ? 64 : TMEM_NEED <= 128 ? 128
                                 : TMEM_NEED <= 256 ? 256 : 512;
  constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) |
                             ((uint32_t)(TC_BM >> 4) << 24);
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
  uint8_t* Bh = smem;
  uint8_t* Bl = smem + B_BYTES;
  uint8_t* As = smem + 2 * B_BYTES;                 // [2 stages][hi 16KB | lo 16KB]
  __shared__ uint64_t tma_bar[2], mma_bar[2];
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
    mbar_init(&tma_bar[0], 1);
    mbar_init(&tma_bar[1], 1);
    mbar_init(&mma_bar[0], 1);
    mbar_init(&mma_bar[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(&tmA) : "memory");
  }
  // B -> hi/lo tiles in the swizzled K-major layout (rows >= n_real are zero)
  for (int idx = tid; idx < N * (K / 4); idx += TC_THREADS) {
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
  auto chunk_coords = [&](int64_t g, int& kcol, int& mrow) {
    const int64_t t = first + (g / KCH) * gridDim.x;
    kcol = (int)(g % KCH) * TC_KC;
    mrow = (int)(t * TC_BM);
  };
  if (tid == 0 && nchunks > 0) {
    int kcol, mrow;
    chunk_coords(0, kcol, mrow);
    mbar_expect_tx(&tma_bar[0], A_STAGE);
    tma_load_2d(As, &tmA, &tma_bar[0], kcol, mrow);
  }
  for (int64_t g = 0; g < nchunks; ++g) {
    const int s = (int)(g & 1);
    const int kc = (int)(g % KCH);
    if (tid == 0 && g + 1 < nchunks) {
      // stage s^1 held chunk g-1: its MMAs must be done before it is overwritten
      if (g >= 1) mbar_wait(&mma_bar[s ^ 1], (uint32_t)(((g - 1) >> 1) & 1));
      int kcol, mrow;
      chunk_coords(g + 1, kcol, mrow);
      mbar_expect_tx(&tma_bar[s ^ 1], A_STAGE);
      tma_load_2d(As + (s ^ 1) * 2 * A_STAGE, &tmA, &tma_bar[s ^ 1], kcol, mrow);
    }
    mbar_wait(&tma_bar[s], (uint32_t)((g >> 1) & 1));
    uint8_t* Ahi = As + s * 2 * A_STAGE;
    uint8_t* Alo = Ahi + A_STAGE;
#pragma unroll 4
    for (int i = tid; i < A_STAGE / 16; i += TC_THREADS) {
      float4 hi, lo;
      split4(*reinterpret_cast<const float4*>(Ahi + i * 16), hi, lo);
      *reinterpret_cast<float4*>(Ahi + i * 16) = hi;
      *reinterpret_cast<float4*>(Alo + i * 16) = lo;
    }
    fence_proxy_async();
    tc_fence_before();
    __syncthreads();
    if (tid == 0) {
      tc_fence_after();
      const uint32_t ah = s_addr(Ahi), al = s_addr(Alo);
      const uint32_t bh = s_addr(Bh + kc * N * 128), bl = s_addr(Bl + kc * N * 128);
      const int grp = kc < NG ? kc : NG - 1;
      const uint32_t tacc = tmem + (uint32_t)(grp * N);
#pragma unroll
      for (int ks = 0; ks < TC_KC / 8; ++ks) {  // K = 8 tf32 (32 bytes) per MMA
        const uint32_t o = ks * 32;
        const uint32_t acc0 = (kc > grp || ks > 0) ? 1u : 0u;  // first MMA of the group
        mma_tf32(tacc, sw128_desc(ah + o), sw128_desc(bh + o), IDESC, acc0);
        mma_tf32(tacc, sw128_desc(ah + o), sw128_desc(bl + o), IDESC, 1u);
        mma_tf32(tacc, sw128_desc(al + o), sw128_desc(bh + o), IDESC, 1u);
      }
      mma_commit(&mma_bar[s]);
    }
    if (kc == KCH - 1) {
      // tile complete: epilogue from TMEM (all MMAs of the tile precede this commit)
      mbar_wait(&mma_bar[s], (uint32_t)((g >> 1) & 1));
      tc_fence_after();
      const int64_t t = first + (g / KCH) * gridDim.x;
      const int64_t row = t * TC_BM + warp * 32 + lane;
      const uint32_t tbase = tmem + ((uint32_t)(warp * 32) << 16);
#pragma unroll 1
      for (int c0 = 0; c0 < N; c0 += 16) {
        float v[16];
        tmem_ld16(tbase + c0, v);
#pragma unroll
        for (int gi = 1; gi < NG; ++gi) {
          float w2[16];
          tmem_ld16(tbase + (uint32_t)(gi * N) + c0, w2);
#pragma unroll
          for (int x = 0; x < 16; ++x) v[x] += w2[x];
        }
        if (row < M) {
#pragma unroll
          for (int j = 0; j < 16; j += 4) {
            const int c = c0 + j;
            const float4 q = make_float4(v[j], v[j + 1], v[j + 2], v[j + 3]);
            if (c + 3 < out.n_split && (out.n_split & 3) == 0) {
              if (out.C0) st4(out.C0 + row * out.n_split + c, q);
              if (out.Cact) st4(out.Cact + row * out.n_split + c, act_fwd4(out.act, q));
            } else if (c < out.n_split) {
#pragma unroll
              for (int x = 0; x < 4; ++x) {
                if (c + x < out.n_split) {
                  if (out.C0) out.C0[row * out.n_split + c + x] = v[j + x];
                  if (out.Cact) out.Cact[row * out.n_split + c + x] = act_fwd(out.act, v[j + x]);
                } else if (c + x < out.n_store) {
                  out.C1[row * (out.n_store - out.n_split) + (c + x - out.n_split)] = v[j + x];
                }
              }
            } else if (c < out.n_store) {
              const int w1 = out.n_store - out.n_split;
#pragma unroll
              for (int x = 0; x < 4; ++x)
                if (c + x < out.n_store) out.C1[row * w1 + (c + x - out.n_split)] = v[j + x];
            }
          }
        }
      }
      tc_fence_before();
      __syncthreads();  // TMEM reads done before the next tile's first MMA
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
// slab of rows: TMA brings 32-row chunks of A and B (128B-swizzled, MN-major
// atoms of 8 rows x 32 columns), threads split them 3xTF32, thread 0 issues
// the MMAs; every TN_GROUP chunks the TMEM accumulator is drained into fp32
// registers (one dW row per thread) so the tensor core's per-MMA rounding
// never compounds over more than TN_GROUP * 12 accumulations.
constexpr int TN_ROWS = 32;   // input rows per chunk
constexpr int TN_GROUP = 2;   // chunks per TMEM drain
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
__global__ void __launch_bounds__(TC_THREADS, 1)
gemm_tn_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                  int64_t M, int64_t rows_per_cta, float* __restrict__ part) {
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
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~uintptr_t(1023));
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
      tma_load_2d(base + b * (TN_ROWS * 128), &tmA, &tma_bar[st], b * 32, r);
#pragma unroll
    for (int b = 0; b < N / 32; ++b)
      tma_load_2d(base + 2 * A_BYTES + b * (TN_ROWS * 128), &tmB, &tma_bar[st], b * 32, r);
  };
  if (tid == 0 && nch > 0) issue_tma(0, (int)(G0 & 1));
  for (int64_t g = 0; g < nch; ++g) {
    const int64_t G = G0 + g;
    const int st = (int)(G & 1);
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
    for (int i = tid; i < (A_BYTES + B_BYTES) / 16; i += TC_THREADS) {
      const bool isA = i < A_BYTES / 16;
      const int li = isA ? i : i - A_BYTES / 16;
      uint8_t* hp = isA ? base + li * 16 : base + 2 * A_BYTES + li * 16;
      uint8_t* lp = hp + (isA ? A_BYTES : B_BYTES);
      const int row = (li * 16 / 128) % TN_ROWS;   // 128-byte row inside a 32-row box
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
  float* out = part + slab * K1 * N + (int64_t)tid * N;  // dW row tid of this slab's partial
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

template <int N, int K>
agnn_status launch_tc(const float* A, int64_t M, const float* B, int n_real, const TcOut& o,
                      cudaStream_t s) {
  auto enc = encode_fn();
  if (!enc) return fail(AGNN_ECUDA, "gemm_tc: cuTensorMapEncodeTiled unavailable");
  CUtensorMap map;
  cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)M};
  cuuint64_t strides[1] = {(cuuint64_t)K * 4};
  cuuint32_t box[2] = {(cuuint32_t)TC_KC, (cuuint32_t)TC_BM};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(A), dims, strides,
                   box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(AGNN_ECUDA, "gemm_tc: tensor map encode failed");
  constexpr int smem = 2 * (K / TC_KC) * N * 128 + 2 * 2 * TC_BM * 128 + 1024;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(gemm_tc_kernel<N, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  int sms = kNumSMs, dev = 0;
  if (cudaGetDevice(&dev) == cudaSuccess)
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int64_t ntiles = (M + TC_BM - 1) / TC_BM;
  const int grid = (int)std::min<int64_t>(ntiles, sms);
  gemm_tc_kernel<N, K><<<grid, TC_THREADS, smem, s>>>(map, B, n_real, M, o);
  AGNN_LAUNCH_CHECK("gemm_tc_kernel");
  return AGNN_OK;
}

bool map_rows_box32(CUtensorMap* map, const float* base, int64_t rows, int cols) {
  auto enc = encode_fn();
  if (!enc) return false;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)cols * 4};
  cuuint32_t box[2] = {32, (cuuint32_t)TN_ROWS};
  cuuint32_t es[2] = {1, 1};
  return enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box,
             es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B,
             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

__global__ void tn_sum_kernel(const float* __restrict__ part, int splits, int64_t count,
                              float* __restrict__ C) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= count) return;
  double s = 0.0;  // fixed order, fp64 across the slab partials
  for (int p = 0; p < splits; ++p) s += (double)part[(int64_t)p * count + i];
  C[i] = (float)s;
}

template <int K1, int N>
agnn_status launch_tn_tc(const float* A, int64_t M, const float* B, float* C, float* ws,
                         cudaStream_t s) {
  CUtensorMap ma, mb;
  if (!map_rows_box32(&ma, A, M, K1) || !map_rows_box32(&mb, B, M, N))
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
  // slabs of >= 8192 rows, at most kTnMaxSlabs of them; each slab leaves one fp32 partial
  int64_t rps = (M + kTnMaxSlabs - 1) / kTnMaxSlabs;
  rps = std::max<int64_t>(rps, 8192);
  rps = (rps + TN_ROWS - 1) / TN_ROWS * TN_ROWS;
  const int64_t nslabs = (M + rps - 1) / rps;
  const int grid = (int)std::min<int64_t>(nslabs, sms);
  gemm_tn_tc_kernel<K1, N><<<grid, TC_THREADS, smem, s>>>(ma, mb, M, rps, ws);
  AGNN_LAUNCH_CHECK("gemm_tn_kernel");
  const int64_t cnt = (int64_t)K1 * N;
  tn_sum_kernel<<<(unsigned)((cnt + 255) / 256), 256, 0, s>>>(ws, (int)nslabs, cnt, C);
  AGNN_LAUNCH_CHECK("sum_splits_kernel");
  return AGNN_OK;
}

bool tc_disabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("AGNN_GEMM");
    v = (e && std::string(e) == "simt") ? 1 : 0;
  }
  return v == 1;
}

template <int K1, int N>
agnn_status launch_tn_tc(const float* A, int64_t M, const float* B, float* C, float* ws,
                         cudaStream_t s);

}  // namespace

// C[K1 x N] = A^T B over M rows on tensor cores (K1 = 128, N in {64, 128}); ws holds
// one K1 x N partial per SM.  AGNN_EUNSUPPORTED for other shapes.
agnn_status gemm_tn_tc(const float* A, int64_t M, int K1, const float* B, int N, float* C,
                       float* ws, cudaStream_t s) {
  if (tc_disabled() || M <= 0) return AGNN_EUNSUPPORTED;
  if ((reinterpret_cast<uintptr_t>(A) & 15) || (reinterpret_cast<uintptr_t>(B) & 15))
    return AGNN_EUNSUPPORTED;
  if (K1 == 128 && N == 128) return launch_tn_tc<128, 128>(A, M, B, C, ws, s);
  if (K1 == 128 && N == 64) return launch_tn_tc<128, 64>(A, M, B, C, ws, s);
  return AGNN_EUNSUPPORTED;
}

// C = A * B^T with B [n_real x K] K-major; columns padded to N_pad (multiple of 16).
// Returns AGNN_EUNSUPPORTED when the shape has no tcgen05 instantiation.
agnn_status gemm_tc(const float* A, int64_t M, int K, const float* B, int n_real, float* C0,
                    int n_split, float* C1, int n_store, float* Cact, int act, cudaStream_t s) {
  if (tc_disabled()) return AGNN_EUNSUPPORTED;
  if (M <= 0) return AGNN_OK;
  if ((reinterpret_cast<uintptr_t>(A) & 15) || (K % 32)) return AGNN_EUNSUPPORTED;
  TcOut o{C0, C1, Cact, n_split, n_store, act};
  const int npad = (n_real + 15) / 16 * 16;
  if (K == 128 && npad == 128) return launch_tc<128, 128>(A, M, B, n_real, o, s);
  if (K == 128 && npad == 144) return launch_tc<144, 128>(A, M, B, n_real, o, s);
  if (K == 128 && npad == 160) return launch_tc<160, 128>(A, M, B, n_real, o, s);
  if (K == 64 && npad == 64) return launch_tc<64, 64>(A, M, B, n_real, o, s);
  if (K == 64 && npad == 80) return launch_tc<80, 64>(A, M, B, n_real, o, s);
  if (K == 64 && npad == 128) return launch_tc<128, 64>(A, M, B, n_real, o, s);
  if (K == 128 && npad == 64) return launch_tc<64, 128>(A, M, B, n_real, o, s);
  return AGNN_EUNSUPPORTED;
}

}  // namespace agnn
