// Probe: TMA tile::gather4 vs LDG.128 vs LDGSTS for random 512-byte row gathers on B200.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* b, int cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(cnt));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t phase) {
  asm volatile(
      "{\n.reg .pred p;\nWAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n}\n" ::"r"(sa(b)), "r"(phase) : "memory");
}
__device__ __forceinline__ void tma_gather4(void* dst, const CUtensorMap* map, uint64_t* bar, int col,
                                            int r0, int r1, int r2, int r3) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4, %5, %6, %7}], [%2];"
      ::"r"(sa(dst)), "l"(map), "r"(sa(bar)), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3)
      : "memory");
}

// each warp: `per_warp` gathers of 4 rows; ring of S stages, one mbarrier per stage
template <int S>
__global__ void __launch_bounds__(256) k_tma(const __grid_constant__ CUtensorMap map, const int* idx,
                                              long per_warp, float* out) {
  extern __shared__ __align__(1024) unsigned char smem[];
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float4* ring = (float4*)(smem + w * S * 2048);
  __shared__ uint64_t bars[8][S];
  if (lane == 0) for (int s = 0; s < S; ++s) mbar_init(&bars[w][s], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const long gw = (blockIdx.x * (long)blockDim.x + threadIdx.x) >> 5;
  const int* my = idx + gw * per_warp * 4;
  float4 acc = make_float4(0, 0, 0, 0);
  auto issue = [&](long g) {
    const int s = g % S;
    if (lane == 0) {
      mbar_expect_tx(&bars[w][s], 2048);
      tma_gather4(ring + s * 128, &map, &bars[w][s], 0, my[4 * g], my[4 * g + 1], my[4 * g + 2], my[4 * g + 3]);
    }
  };
  long g = 0;
  for (; g < S - 1 && g < per_warp; ++g) issue(g);
  for (long c = 0; c < per_warp; ++c) {
    const int s = c % S;
    mbar_wait(&bars[w][s], (c / S) & 1);
    #pragma unroll
    for (int r = 0; r < 4; ++r) {
      float4 v = ring[s * 128 + r * 32 + lane];
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    __syncwarp();
    if (g < per_warp) { issue(g); ++g; }
  }
  out[gw * 32 + lane] = acc.x + acc.y + acc.z + acc.w;
}

template <int U>
__global__ void __launch_bounds__(256) k_ldg(const float4* table, const int* idx, long per_warp, float* out) {
  const int lane = threadIdx.x & 31;
  const long gw = (blockIdx.x * (long)blockDim.x + threadIdx.x) >> 5;
  const int* my = idx + gw * per_warp * 4;
  float4 acc = make_float4(0, 0, 0, 0);
  for (long e = 0; e < per_warp * 4; e += U) {
    float4 v[U];
    #pragma unroll
    for (int u = 0; u < U; ++u) v[u] = __ldg(table + (long)my[e + u] * 32 + lane);
    #pragma unroll
    for (int u = 0; u < U; ++u) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
  }
  out[gw * 32 + lane] = acc.x + acc.y + acc.z + acc.w;
}

int main() {
  const long n = 1L << 24, K = 128;
  const long warps = 148L * 64, per_warp = 2048;  // gathers of 4 rows per warp
  const long total_rows = warps * per_warp * 4;
  float* table;
  int* idx;
  float* out;
  CK(cudaMalloc(&table, n * K * 4));
  CK(cudaMalloc(&idx, total_rows * 4));
  CK(cudaMalloc(&out, warps * 32 * 4));
  std::vector<float> ht(n * K);
  for (long i = 0; i < n * K; ++i) ht[i] = (float)((i * 2654435761u) % 1000) * 1e-3f;
  CK(cudaMemcpy(table, ht.data(), n * K * 4, cudaMemcpyHostToDevice));
  std::vector<int> hi(total_rows);
  unsigned long long x = 88172645463325252ull;
  for (long i = 0; i < total_rows; ++i) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; hi[i] = (int)(x % n); }
  CK(cudaMemcpy(idx, hi.data(), total_rows * 4, cudaMemcpyHostToDevice));

  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q));
  CUtensorMap map;
  for (int boxrows : {1}) {
    cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)n};
    cuuint64_t strides[1] = {(cuuint64_t)K * 4};
    cuuint32_t box[2] = {(cuuint32_t)K, (cuuint32_t)boxrows};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, table, dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode boxrows=%d -> %d\n", boxrows, (int)r);
    if (r != CUDA_SUCCESS) continue;
    constexpr int S = 4;
    const int smem = 8 * S * 2048;
    CK(cudaFuncSetAttribute(k_tma<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    CK(cudaFuncSetAttribute(k_tma<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 2 * 2048));
    CK(cudaFuncSetAttribute(k_tma<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, 8 * 8 * 2048));
    // correctness on a small launch
    k_tma<S><<<1, 32, smem>>>(map, idx, 4, out);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("tma launch failed: %s\n", cudaGetErrorString(e)); return 1; }
    std::vector<float> ho(32);
    CK(cudaMemcpy(ho.data(), out, 32 * 4, cudaMemcpyDeviceToHost));
    double maxerr = 0;
    for (int l = 0; l < 32; ++l) {
      double ref = 0;
      for (int g = 0; g < 16; ++g) for (int c = 0; c < 4; ++c) ref += ht[(long)hi[g] * K + l * 4 + c];
      maxerr = std::max(maxerr, std::abs(ref - ho[l]));
    }
    printf("  gather4 correctness max err %.3g\n", maxerr);
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(a);
      k_tma<S><<<warps / 8, 256, smem>>>(map, idx, per_warp, out);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      float ms; cudaEventElapsedTime(&ms, a, b);
      printf("  tma gather4 S=%d: %.3f ms, %.1f GB/s (rows)\n", S, ms, total_rows * 512.0 / ms / 1e6);
    }
    for (int rep = 0; rep < 2; ++rep) {
      cudaEventRecord(a);
      k_tma<2><<<warps / 8, 256, 8 * 2 * 2048>>>(map, idx, per_warp, out);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      float ms; cudaEventElapsedTime(&ms, a, b);
      printf("  tma gather4 S=2: %.3f ms, %.1f GB/s (rows)\n", ms, total_rows * 512.0 / ms / 1e6);
      cudaEventRecord(a);
      k_tma<8><<<warps / 8, 256, 8 * 8 * 2048>>>(map, idx, per_warp, out);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      cudaEventElapsedTime(&ms, a, b);
      printf("  tma gather4 S=8: %.3f ms, %.1f GB/s (rows)\n", ms, total_rows * 512.0 / ms / 1e6);
    }
  }
  for (int rep = 0; rep < 2; ++rep) {
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    cudaEventRecord(a);
    k_ldg<8><<<warps / 8, 256>>>((const float4*)table, idx, per_warp, out);
    cudaEventRecord(b);
    CK(cudaEventSynchronize(b));
    float ms; cudaEventElapsedTime(&ms, a, b);
    printf("ldg U=8 (64 warps/SM): %.3f ms, %.1f GB/s\n", ms, total_rows * 512.0 / ms / 1e6);
    cudaEventRecord(a);
    k_ldg<4><<<warps / 8, 256>>>((const float4*)table, idx, per_warp, out);
    cudaEventRecord(b);
    CK(cudaEventSynchronize(b));
    cudaEventElapsedTime(&ms, a, b);
    printf("ldg U=4 (64 warps/SM): %.3f ms, %.1f GB/s\n", ms, total_rows * 512.0 / ms / 1e6);
    cudaEventRecord(a);
    k_ldg<16><<<warps / 8, 256>>>((const float4*)table, idx, per_warp, out);
    cudaEventRecord(b);
    CK(cudaEventSynchronize(b));
    cudaEventElapsedTime(&ms, a, b);
    printf("ldg U=16 (64 warps/SM): %.3f ms, %.1f GB/s\n", ms, total_rows * 512.0 / ms / 1e6);
  }
  return 0;
}
