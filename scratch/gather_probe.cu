// gather_probe.cu — practical HBM rate of random row gathers on one B200 (the
// access pattern of the GAT sparse kernels): a warp reads whole rows of a large
// table (16 B per lane, one row per warp instruction) at uniformly random row ids.
// Reports GB/s for row sizes 512 B (fp32, k' = 128) and 256 B (bf16), and for
// sequential row ids (a streaming read) as the reference.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_probe gather_probe.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

__global__ void fill_idx(uint32_t* idx, int64_t m, uint32_t rows, int random) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m;
       i += (int64_t)gridDim.x * blockDim.x) {
    uint64_t x = (uint64_t)i * 0x9E3779B97F4A7C15ull + 0x632BE59BD9B4E019ull;
    x ^= x >> 31; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 29;
    idx[i] = random ? (uint32_t)(x % rows) : (uint32_t)(i % rows);
  }
}

// LPR lanes per row (16 B each): 32 = 512-byte rows, 16 = 256-byte rows (two rows
// per warp instruction); U rows in flight per lane group
template <int LPR, int U>
__global__ void __launch_bounds__(256) gather(const float4* __restrict__ tab,
                                              const uint32_t* __restrict__ idx, int64_t m,
                                              float* __restrict__ out) {
  const int lane = threadIdx.x & 31, sub = lane / LPR, q = lane % LPR;
  constexpr int RPW = 32 / LPR;  // rows per warp instruction
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (int64_t b = gw * 32; b < m; b += nw * 32) {
    const uint32_t my = b + lane < m ? idx[b + lane] : 0;
#pragma unroll
    for (int k0 = 0; k0 < 32; k0 += RPW * U) {
      float4 v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const uint32_t r = __shfl_sync(0xffffffffu, my, k0 + u * RPW + sub);
        v[u] = __ldg(tab + (int64_t)r * LPR + q);
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w;
      }
    }
  }
  out[((int64_t)blockIdx.x * blockDim.x + threadIdx.x)] = acc.x + acc.y + acc.z + acc.w;
}

template <int LPR, int U>
double run(const float4* tab, const uint32_t* idx, int64_t m, float* out, int blocks) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  gather<LPR, U><<<blocks, 256>>>(tab, idx, m, out);
  cudaEventRecord(a);
  const int reps = 5;
  for (int r = 0; r < reps; ++r) gather<LPR, U><<<blocks, 256>>>(tab, idx, m, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  return (double)m * LPR * 16 * reps / (ms * 1e-3) / 1e9;
}

int main() {
  const int64_t table_bytes = 8LL << 30;  // 8 GiB table (>> 126 MB L2)
  const int64_t m = 1LL << 28;            // 268M gathers per launch
  float4* tab;
  uint32_t* idx;
  float* out;
  cudaMalloc(&tab, table_bytes);
  // non-zero, varied contents (no reliance on zero pages)
  fill_idx<<<148 * 8, 256>>>(reinterpret_cast<uint32_t*>(tab), table_bytes / 4, 0xffffffffu, 1);
  cudaMalloc(&idx, m * 4);
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int blocks = sms * 8;
  cudaMalloc(&out, (size_t)blocks * 256 * 4);
  for (int random = 1; random >= 0; --random) {
    for (int rb : {512, 256}) {
      const uint32_t rows = (uint32_t)(table_bytes / rb);
      fill_idx<<<sms * 8, 256>>>(idx, m, rows, random);
      cudaDeviceSynchronize();
      for (int bps : {2, 3, 8}) {  // resident 256-thread blocks per SM (16, 24, 64 warps)
        const int nb = sms * bps;
        double g4 = rb == 512 ? run<32, 4>(tab, idx, m, out, nb) : run<16, 4>(tab, idx, m, out, nb);
        double g8 = rb == 512 ? run<32, 8>(tab, idx, m, out, nb) : run<16, 8>(tab, idx, m, out, nb);
        double g16 = rb == 512 ? run<32, 16>(tab, idx, m, out, nb) : run<16, 16>(tab, idx, m, out, nb);
        printf("%s rows of %d B, %2d warps/SM: %5.0f GB/s (4 rows in flight / lane group), %5.0f (8), %5.0f (16)\n",
               random ? "random    " : "sequential", rb, bps * 8, g4, g8, g16);
      }
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("error: %s\n", cudaGetErrorString(e));
  return 0;
}
