// gather_probe_v8.cu — random 1 KB row gathers (k = 256 fp32, the C4 rows): two
// 16-byte loads per lane per row (the av_batched layout, V = 2) against one 32-byte
// load per lane (ld.global.nc.v8.f32, sm_100), and 512-byte rows with 16 B per lane
// against 32 B per lane on half-warps (two rows per instruction).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_probe_v8 gather_probe_v8.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void fill_idx(uint32_t* idx, int64_t m, uint32_t rows) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t x = (uint64_t)i * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull;
    x ^= x >> 31; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 29;
    idx[i] = (uint32_t)(x % rows);
  }
}
__device__ __forceinline__ void ld8(const float* p, float (&r)[8]) {
  asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(r[0]), "=f"(r[1]), "=f"(r[2]), "=f"(r[3]), "=f"(r[4]), "=f"(r[5]),
                 "=f"(r[6]), "=f"(r[7])
               : "l"(p));
}
// MODE 0: ROWB-byte rows, 16 B per lane loads (ROWB/512 loads per lane per row)
// MODE 1: ROWB-byte rows, 32 B per lane loads (ROWB/1024 loads per lane per row,
//         ROWB = 512: two rows per instruction on half-warps)
template <int MODE, int ROWB, int U>
__global__ void __launch_bounds__(256) gather(const float* __restrict__ tab,
                                              const uint32_t* __restrict__ idx, int64_t m,
                                              float* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  constexpr int RF = ROWB / 4;  // floats per row
  float acc = 0.f;
  for (int64_t b = gw * 32; b < m; b += nw * 32) {
    const uint32_t my = b + lane < m ? idx[b + lane] : 0;
    if (MODE == 0) {
      constexpr int L = ROWB / 512;  // 16-byte loads per lane per row
#pragma unroll
      for (int k0 = 0; k0 < 32; k0 += U) {
        float4 v[U][L];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const uint32_t r = __shfl_sync(0xffffffffu, my, k0 + u);
#pragma unroll
          for (int l = 0; l < L; ++l)
            v[u][l] = __ldg(reinterpret_cast<const float4*>(tab + (int64_t)r * RF + l * 128) + lane);
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int l = 0; l < L; ++l) acc += v[u][l].x + v[u][l].y + v[u][l].z + v[u][l].w;
      }
    } else {
      constexpr int LPR = ROWB / 32;   // lanes per row at 32 B each
      constexpr int RPI = 32 / LPR;    // rows per instruction
      const int sub = lane / LPR, q = lane % LPR;
#pragma unroll
      for (int k0 = 0; k0 < 32; k0 += U * RPI) {
        float v[U][8];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const uint32_t r = __shfl_sync(0xffffffffu, my, k0 + u * RPI + sub);
          ld8(tab + (int64_t)r * RF + q * 8, v[u]);
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int c = 0; c < 8; ++c) acc += v[u][c];
      }
    }
  }
  out[((int64_t)blockIdx.x * blockDim.x + threadIdx.x)] = acc;
}

template <int MODE, int ROWB, int U>
double run(const float* tab, const uint32_t* idx, int64_t m, float* out, int blocks) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  gather<MODE, ROWB, U><<<blocks, 256>>>(tab, idx, m, out);
  cudaEventRecord(a);
  const int reps = 5;
  for (int r = 0; r < reps; ++r) gather<MODE, ROWB, U><<<blocks, 256>>>(tab, idx, m, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  return (double)m * ROWB * reps / (ms * 1e-3) / 1e9;
}

int main() {
  const int64_t table_bytes = 8LL << 30;
  const int64_t m = 1LL << 26;
  float* tab;
  uint32_t* idx;
  float* out;
  cudaMalloc(&tab, table_bytes);
  cudaMemset(tab, 1, table_bytes);
  cudaMalloc(&out, (size_t)148 * 8 * 256 * 4);
  cudaMalloc(&idx, m * 4);
  for (int wps : {16, 24}) {
    const int blocks = 148 * wps / 8;
    fill_idx<<<148 * 8, 256>>>(idx, m, (uint32_t)(table_bytes / 1024));
    cudaDeviceSynchronize();
    printf("%d warps/SM, 1 KB rows:  2x16B/lane U=2 %6.0f U=4 %6.0f | 1x32B/lane U=2 %6.0f U=4 %6.0f GB/s\n",
           wps, run<0, 1024, 2>(tab, idx, m, out, blocks), run<0, 1024, 4>(tab, idx, m, out, blocks),
           run<1, 1024, 2>(tab, idx, m, out, blocks), run<1, 1024, 4>(tab, idx, m, out, blocks));
    fill_idx<<<148 * 8, 256>>>(idx, m, (uint32_t)(table_bytes / 512));
    cudaDeviceSynchronize();
    printf("%d warps/SM, 512 B rows: 1x16B/lane U=4 %6.0f U=8 %6.0f | 32B/lane pairs U=2 %6.0f U=4 %6.0f GB/s\n",
           wps, run<0, 512, 4>(tab, idx, m, out, blocks), run<0, 512, 8>(tab, idx, m, out, blocks),
           run<1, 512, 2>(tab, idx, m, out, blocks), run<1, 512, 4>(tab, idx, m, out, blocks));
  }
  return 0;
}
