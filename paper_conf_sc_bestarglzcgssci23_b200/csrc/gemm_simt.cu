// gemm_simt.cu — fp32 FFMA GEMMs for the dense projections (PAPER.md:141 H' = HW,
// :149 MM) and the weight gradient (Eq. 5, Y = H^T ... G).
//
// Exact fp32 arithmetic (one rounding per FMA), 128x128 block tiles, 8x8 register
// micro-tiles, register-prefetched 8-deep K slices.  These are the fp32-accurate
// path; the tcgen05 3xTF32 GEMM (gemm_tc.cu) replaces gemm_rows where enabled.
#include <algorithm>

#include "internal.cuh"

namespace agnn {
namespace {

constexpr int BM = 128, BN = 128, BK = 8, TPB = 256;

// C = A * op(B) over one 128x128 tile.
__global__ void __launch_bounds__(TPB)
gemm_rows_kernel(const float* __restrict__ A, int64_t M, int K, const float* __restrict__ B,
                 int b_trans, int N, float* __restrict__ C0, int n_split, float* __restrict__ C1,
                 float* __restrict__ Cact, int act, int n_store) {
  __shared__ __align__(16) float As[2][BK][BM + 4];
  __shared__ __align__(16) float Bs[2][BK][BN + 4];
  const int tid = threadIdx.x, tx = tid % 16, ty = tid / 16;
  const int64_t m0 = (int64_t)blockIdx.x * BM;
  const int n0 = blockIdx.y * BN;

  // loader mapping: A tile 128 x 8 -> thread loads rows (tid/2), cols (tid%2)*4..+3
  const int a_r = tid / 2, a_c = (tid % 2) * 4;
  // B tile 8 x 128: non-trans thread loads row tid/32, cols (tid%32)*4; trans: n = tid/2, k = (tid%2)*4
  auto load_a = [&](int k0) -> float4 {
    const int64_t r = m0 + a_r;
    if (r < M && k0 + a_c < K) return ldg4(A + r * K + k0 + a_c);
    return f4(0.f);
  };
  auto load_b = [&](int k0) -> float4 {
    if (!b_trans) {
      const int kr = k0 + tid / 32, c = n0 + (tid % 32) * 4;
      if (kr < K && c < N) return ldg4(B + (int64_t)kr * N + c);
    } else {
      const int c = n0 + tid / 2, kr = k0 + (tid % 2) * 4;
      if (c < N && kr < K) return ldg4(B + (int64_t)c * K + kr);
    }
    return f4(0.f);
  };
  auto store_tiles = [&](int buf, float4 av, float4 bv) {
    As[buf][a_c + 0][a_r] = av.x;
    As[buf][a_c + 1][a_r] = av.y;
    As[buf][a_c + 2][a_r] = av.z;
    As[buf][a_c + 3][a_r] = av.w;
    if (!b_trans) {
      *reinterpret_cast<float4*>(&Bs[buf][tid / 32][(tid % 32) * 4]) = bv;
    } else {
      const int c = tid / 2, kr = (tid % 2) * 4;
      Bs[buf][kr + 0][c] = bv.x;
      Bs[buf][kr + 1][c] = bv.y;
      Bs[buf][kr + 2][c] = bv.z;
      Bs[buf][kr + 3][c] = bv.w;
    }
  };

  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;

  float4 av = load_a(0), bv = load_b(0);
  store_tiles(0, av, bv);
  __syncthreads();
  int buf = 0;
  for (int k0 = 0; k0 < K; k0 += BK) {
    const bool more = k0 + BK < K;
    if (more) {
      av = load_a(k0 + BK);
      bv = load_b(k0 + BK);
    }
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      const float4 a0 = *reinterpret_cast<const float4*>(&As[buf][kk][ty * 4]);
      const float4 a1 = *reinterpret_cast<const float4*>(&As[buf][kk][64 + ty * 4]);
      const float4 b0 = *reinterpret_cast<const float4*>(&Bs[buf][kk][tx * 4]);
      const float4 b1 = *reinterpret_cast<const float4*>(&Bs[buf][kk][64 + tx * 4]);
      const float ar[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
      const float br[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(ar[i], br[j], acc[i][j]);
    }
    if (more) {
      store_tiles(buf ^ 1, av, bv);
      __syncthreads();
      buf ^= 1;
    }
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int64_t r = m0 + (i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4);
    if (r >= M) continue;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int c = n0 + (j < 4 ? tx * 4 + j : 64 + tx * 4 + j - 4);
      if (c >= n_store) continue;
      if (c < n_split) {
        if (C0) C0[r * n_split + c] = acc[i][j];
        if (Cact) Cact[r * n_split + c] = act_fwd(act, acc[i][j]);
      } else {
        C1[r * (n_store - n_split) + (c - n_split)] = acc[i][j];
      }
    }
  }
}

int tn_splits(int K1, int N) {
  const int tiles = ((K1 + BM - 1) / BM) * ((N + BN - 1) / BN);
  const int s = (2 * kNumSMs) / tiles;
  return s < 1 ? 1 : s;
}

// partial[split] = A[rows of split]^T B[rows of split] for one 128x128 output tile
__global__ void __launch_bounds__(TPB)
gemm_tn_kernel(const float* __restrict__ A, int64_t M, int K1, const float* __restrict__ B, int N,
               float* __restrict__ part, int64_t rows_per_split) {
  __shared__ __align__(16) float As[2][BK][BM + 4];
  __shared__ __align__(16) float Bs[2][BK][BN + 4];
  const int tid = threadIdx.x, tx = tid % 16, ty = tid / 16;
  const int tiles_n = (N + BN - 1) / BN;
  const int r0 = (blockIdx.x / tiles_n) * BM, c0 = (blockIdx.x % tiles_n) * BN;
  const int64_t m_beg = (int64_t)blockIdx.y * rows_per_split;
  const int64_t m_end = min(M, m_beg + rows_per_split);
  // loaders: 8 rows x 128 cols each from A (cols r0..) and B (cols c0..)
  const int lr = tid / 32, lc = (tid % 32) * 4;
  auto ld = [&](const float* X, int W, int col0, int64_t m) -> float4 {
    if (m < m_end && col0 + lc < W) return ldg4(X + m * W + col0 + lc);
    return f4(0.f);
  };
  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
  if (m_beg < m_end) {
    float4 av = ld(A, K1, r0, m_beg + lr), bv = ld(B, N, c0, m_beg + lr);
    *reinterpret_cast<float4*>(&As[0][lr][lc]) = av;
    *reinterpret_cast<float4*>(&Bs[0][lr][lc]) = bv;
    __syncthreads();
    int buf = 0;
    for (int64_t m = m_beg; m < m_end; m += BK) {
      const bool more = m + BK < m_end;
      if (more) {
        av = ld(A, K1, r0, m + BK + lr);
        bv = ld(B, N, c0, m + BK + lr);
      }
#pragma unroll
      for (int kk = 0; kk < BK; ++kk) {
        const float4 a0 = *reinterpret_cast<const float4*>(&As[buf][kk][ty * 4]);
        const float4 a1 = *reinterpret_cast<const float4*>(&As[buf][kk][64 + ty * 4]);
        const float4 b0 = *reinterpret_cast<const float4*>(&Bs[buf][kk][tx * 4]);
        const float4 b1 = *reinterpret_cast<const float4*>(&Bs[buf][kk][64 + tx * 4]);
        const float ar[8] = {a0.x, a0.y, a0.z, a0.w, a1.x, a1.y, a1.z, a1.w};
        const float br[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
#pragma unroll
        for (int i = 0; i < 8; ++i)
#pragma unroll
          for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(ar[i], br[j], acc[i][j]);
      }
      if (more) {
        *reinterpret_cast<float4*>(&As[buf ^ 1][lr][lc]) = av;
        *reinterpret_cast<float4*>(&Bs[buf ^ 1][lr][lc]) = bv;
        __syncthreads();
        buf ^= 1;
      }
    }
  }
  float* P = part + (int64_t)blockIdx.y * K1 * N;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int r = r0 + (i < 4 ? ty * 4 + i : 64 + ty * 4 + i - 4);
    if (r >= K1) continue;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int c = c0 + (j < 4 ? tx * 4 + j : 64 + tx * 4 + j - 4);
      if (c < N) P[(int64_t)r * N + c] = acc[i][j];
    }
  }
}

__global__ void transpose_kernel(const float* __restrict__ X, int rows, int cols,
                                 float* __restrict__ Y) {
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < rows * cols; i += gridDim.x * blockDim.x)
    Y[(i % cols) * rows + i / cols] = X[i];
}

__global__ void sum_splits_kernel(const float* __restrict__ part, int splits, int64_t count,
                                  float* __restrict__ C) {
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= count) return;
  double s = 0.0;  // fixed order, fp64 across the split partials
  for (int p = 0; p < splits; ++p) s += (double)part[(int64_t)p * count + i];
  C[i] = (float)s;
}

}  // namespace

agnn_status gemm_tc(const float* A, int64_t M, int K, const float* B, int n_real, float* C0,
                    int n_split, float* C1, int n_store, float* Cact, int act, cudaStream_t s,
                    bf16* C0h = nullptr, const PeerOut* peers = nullptr);

namespace {
// Y[i] = bf16_rn(X[i]) over rows x cols (cols % 4 == 0)
__global__ void to_bf16_kernel(const float* __restrict__ X, int64_t count4, bf16* __restrict__ Y) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count4;
       i += (int64_t)gridDim.x * blockDim.x)
    st4(Y + 4 * i, ldg4(X + 4 * i));
}
}  // namespace

agnn_status gemm_rows_bf16(const float* A, int64_t M, int K, const float* B, int N, bf16* C0h,
                           int n_split, float* C1, float* scratch, cudaStream_t s) {
  if (M <= 0) return AGNN_OK;
  agnn_status st = gemm_tc(A, M, K, B, N, nullptr, n_split, C1, N, nullptr, 0, s, C0h);
  if (st != AGNN_EUNSUPPORTED) return st;
  // no tcgen05 instantiation for this shape: fp32 product into scratch, then round
  // (B has (N + 3) / 4 * 4 rows, the padding rows zero; columns >= N are not stored)
  if ((st = gemm_rows(A, M, K, B, true, (N + 3) / 4 * 4, scratch, n_split, C1, s, nullptr, 0, N)) !=
      AGNN_OK)
    return st;
  const int64_t c4 = M * n_split / 4;
  to_bf16_kernel<<<(unsigned)std::min<int64_t>((c4 + 255) / 256, kNumSMs * 16), 256, 0, s>>>(
      scratch, c4, C0h);
  AGNN_LAUNCH_CHECK("to_bf16_kernel");
  return AGNN_OK;
}

agnn_status gemm_rows(const float* A, int64_t M, int K, const float* B, bool b_trans, int N,
                      float* C0, int n_split, float* C1, cudaStream_t s, float* Cact, int act,
                      int n_store, const PeerOut* peers, bool* peers_done) {
  if (peers_done) *peers_done = false;
  if (b_trans) {  // tcgen05 3xTF32 path when the shape has an instantiation
    const int ns = (n_store <= 0 || n_store > N) ? N : n_store;
    agnn_status st = gemm_tc(A, M, K, B, ns, C0, n_split, C1, ns, Cact, act, s, nullptr, peers);
    if (st != AGNN_EUNSUPPORTED) {
      if (peers_done) *peers_done = peers != nullptr && st == AGNN_OK;
      return st;
    }
    // no peer epilogue for this shape (the caller pushes the rows instead)
    if (peers && (st = gemm_tc(A, M, K, B, ns, C0, n_split, C1, ns, Cact, act, s)) !=
                     AGNN_EUNSUPPORTED)
      return st;
  }
  if (M <= 0) return AGNN_OK;
  if (K % 4 || N % 4) return fail(AGNN_EINVAL, "gemm_rows: K and N must be multiples of 4");
  dim3 grid((unsigned)((M + BM - 1) / BM), (N + BN - 1) / BN);
  if (n_store <= 0 || n_store > N) n_store = N;
  gemm_rows_kernel<<<grid, TPB, 0, s>>>(A, M, K, B, b_trans ? 1 : 0, N, C0, n_split, C1, Cact,
                                        act, n_store);
  AGNN_LAUNCH_CHECK("gemm_rows_kernel");
  return AGNN_OK;
}

agnn_status transpose(const float* X, int rows, int cols, float* Y, cudaStream_t s) {
  transpose_kernel<<<64, 256, 0, s>>>(X, rows, cols, Y);
  AGNN_LAUNCH_CHECK("transpose_kernel");
  return AGNN_OK;
}

size_t gemm_tn_ws_floats(int K1, int N) {
  const size_t simt = (size_t)tn_splits(K1, N) * K1 * N;
  // one partial per (128 x 128 output block, row slab) (gemm_tn_tc)
  const size_t blocks = (size_t)((K1 + 127) / 128) * ((N + 127) / 128);
  const size_t tc = (size_t)2048 * (K1 < 128 ? K1 : 128) * (N < 128 ? N : 128) * blocks;
  return simt > tc ? simt : tc;
}

agnn_status gemm_tn_tc(const float* A, int64_t M, int K1, const float* B, int N, float* C,
                       float* ws, cudaStream_t s);

agnn_status gemm_tn(const float* A, int64_t M, int K1, const float* B, int N, float* C, float* ws,
                    cudaStream_t s) {
  {
    const agnn_status st = gemm_tn_tc(A, M, K1, B, N, C, ws, s);
    if (st != AGNN_EUNSUPPORTED) return st;
  }
  if (K1 % 4 || N % 4) return fail(AGNN_EINVAL, "gemm_tn: widths must be multiples of 4");
  const int S = tn_splits(K1, N);
  int64_t rps = (M + S - 1) / S;
  rps = (rps + BK - 1) / BK * BK;
  const int tiles = ((K1 + BM - 1) / BM) * ((N + BN - 1) / BN);
  gemm_tn_kernel<<<dim3(tiles, S), TPB, 0, s>>>(A, M, K1, B, N, ws, rps);
  AGNN_LAUNCH_CHECK("gemm_tn_kernel");
  const int64_t cnt = (int64_t)K1 * N;
  sum_splits_kernel<<<(unsigned)((cnt + 255) / 256), 256, 0, s>>>(ws, S, cnt, C);
  AGNN_LAUNCH_CHECK("sum_splits_kernel");
  return AGNN_OK;
}

}  // namespace agnn
