/*
 * libagnngen.so — seeded input generators (host OpenMP + device kernels).
 * Test/bench infrastructure shared by both sides; holds no A-GNN arithmetic.
 * Compiled WITHOUT fast-math so host and device fp32 multiplies agree bit for bit.
 */
#include <cuda_runtime.h>
#include <omp.h>
#include <stdint.h>
#include "agnn_gen.h"

extern "C" {

/* n_samples edge samples of `kind` into src[], dst[] (host). */
int agen_edges_host(int kind, uint64_t seed, int scale, uint64_t n, uint64_t n_samples,
                    uint32_t* src, uint32_t* dst) {
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < (int64_t)n_samples; ++e)
    agen_pair(kind, seed, scale, n, (uint64_t)e, &src[e], &dst[e]);
  return 0;
}

/* out[i] = U[-1,1)(seed, stream, offset + i) * scale (host). */
int agen_fill_host(uint64_t seed, uint64_t stream, uint64_t offset, uint64_t count, float scale,
                   float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < (int64_t)count; ++i)
    out[i] = agen_unif_pm1(seed, stream, offset + (uint64_t)i) * scale;
  return 0;
}

/* rows of a [*, width] tensor: out[r][c] = U[-1,1)(seed, stream, ids[r] * width + c) * scale
 * (host) — the same values agen_fill_host gives at those rows of the whole tensor. */
int agen_fill_rows_host(uint64_t seed, uint64_t stream, const int64_t* ids, int64_t nrows,
                        int64_t width, float scale, float* out) {
#pragma omp parallel for schedule(static)
  for (int64_t r = 0; r < nrows; ++r)
    for (int64_t c = 0; c < width; ++c)
      out[r * width + c] = agen_unif_pm1(seed, stream, (uint64_t)(ids[r] * width + c)) * scale;
  return 0;
}

}  // extern "C"

__global__ void agen_edges_kernel(int kind, uint64_t seed, int scale, uint64_t n, uint64_t n_samples,
                                  uint32_t* __restrict__ src, uint32_t* __restrict__ dst) {
  for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < n_samples;
       e += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t s, d;
    agen_pair(kind, seed, scale, n, e, &s, &d);
    src[e] = s;
    dst[e] = d;
  }
}

__global__ void agen_fill_kernel(uint64_t seed, uint64_t stream, uint64_t offset, uint64_t count,
                                 float scale, float* __restrict__ out) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < count;
       i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = agen_unif_pm1(seed, stream, offset + i) * scale;
}

extern "C" {

/* Device versions: pointers are device pointers, work is enqueued on `stream`. */
int agen_edges_device(int kind, uint64_t seed, int scale, uint64_t n, uint64_t n_samples,
                      uint32_t* src, uint32_t* dst, cudaStream_t stream) {
  if (n_samples == 0) return 0;
  agen_edges_kernel<<<148 * 16, 256, 0, stream>>>(kind, seed, scale, n, n_samples, src, dst);
  return cudaGetLastError() == cudaSuccess ? 0 : 1;
}

int agen_fill_device(uint64_t seed, uint64_t stream_id, uint64_t offset, uint64_t count, float scale,
                     float* out, cudaStream_t stream) {
  if (count == 0) return 0;
  agen_fill_kernel<<<148 * 16, 256, 0, stream>>>(seed, stream_id, offset, count, scale, out);
  return cudaGetLastError() == cudaSuccess ? 0 : 1;
}

}  // extern "C"
