// train.cu — the two steps either side of the layer path in a training loop
// (SURVEY §8(f) f1): the loss of reading A13 and the SGD update of PAPER.md:244.
//
//   L = <R, H^L> = sum_e R_e H_e        (reading A13: dL/dH^L = R, the Eq. 4 bootstrap)
//   W <- W - lr * dW                    ("W^l is updated with the gradient Y^l")
//
// The loss is a deterministic two-stage reduction: a fixed grid of persistent
// blocks writes one fp64 partial per block (fixed-order tree inside the block),
// then one block adds the partials in index order.  Both kernels are
// HBM-bound streams (8 B read per element for the loss, 12 B per element for SGD).
#include "internal.cuh"

namespace agnn {
namespace {

constexpr int kLossThreads = 512;

__device__ __forceinline__ double block_sum(double v, double* red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_down_sync(0xffffffffu, v, o);
  if (lane == 0) red[warp] = v;
  __syncthreads();
  double s = 0.0;
  if (threadIdx.x == 0)
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) s += red[w];
  return s;  // valid in thread 0
}

__global__ void __launch_bounds__(kLossThreads)
loss_partial_kernel(const float* __restrict__ R, const float* __restrict__ H, int64_t count,
                    double* __restrict__ part) {
  __shared__ double red[kLossThreads / 32];
  double acc = 0.0;
  const int64_t n4 = count / 4;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  // 16-byte loads when both bases are aligned (the ABI requires 16-byte alignment)
  for (int64_t i = t0; i < n4; i += stride) {
    const float4 r = ldg4(R + 4 * i), h = ldg4(H + 4 * i);
    acc += (double)r.x * h.x + (double)r.y * h.y + (double)r.z * h.z + (double)r.w * h.w;
  }
  for (int64_t i = 4 * n4 + t0; i < count; i += stride) acc += (double)R[i] * H[i];
  const double s = block_sum(acc, red);
  if (threadIdx.x == 0) part[blockIdx.x] = s;
}

__global__ void __launch_bounds__(kLossThreads)
loss_final_kernel(const double* __restrict__ part, int n, double* __restrict__ loss) {
  __shared__ double red[kLossThreads / 32];
  double acc = 0.0;
  for (int i = threadIdx.x; i < n; i += blockDim.x) acc += part[i];
  const double s = block_sum(acc, red);
  if (threadIdx.x == 0) *loss = s;
}

__global__ void sgd_kernel(float* __restrict__ W, const float* __restrict__ dW, int64_t count,
                           float lr) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
       i += (int64_t)gridDim.x * blockDim.x)
    W[i] = fmaf(-lr, dW[i], W[i]);
}

}  // namespace
}  // namespace agnn

using namespace agnn;

extern "C" agnn_status agnn_loss_inner(const float* R, const float* H, int64_t count,
                                       double* scratch, double* loss, cudaStream_t s) {
  if (count < 0 || !scratch || !loss || (count > 0 && (!R || !H)))
    return fail(AGNN_EINVAL, "agnn_loss_inner: bad arguments");
  if ((reinterpret_cast<uintptr_t>(R) | reinterpret_cast<uintptr_t>(H)) & 15)
    return fail(AGNN_EINVAL, "agnn_loss_inner: R and H must be 16-byte aligned");
  const int blocks = AGNN_LOSS_SCRATCH;  // fixed: the summation order never depends on the GPU
  loss_partial_kernel<<<blocks, kLossThreads, 0, s>>>(R, H, count, scratch);
  AGNN_LAUNCH_CHECK("loss_partial_kernel");
  loss_final_kernel<<<1, kLossThreads, 0, s>>>(scratch, blocks, loss);
  AGNN_LAUNCH_CHECK("loss_final_kernel");
  return AGNN_OK;
}

extern "C" agnn_status agnn_sgd_step(float* W, const float* dW, int64_t count, float lr,
                                     cudaStream_t s) {
  if (count < 0 || (count > 0 && (!W || !dW))) return fail(AGNN_EINVAL, "agnn_sgd_step: bad arguments");
  if (count == 0) return AGNN_OK;
  const int64_t blocks = std::min<int64_t>((count + 255) / 256, (int64_t)kNumSMs * 16);
  sgd_kernel<<<(unsigned)blocks, 256, 0, s>>>(W, dW, count, lr);
  AGNN_LAUNCH_CHECK("sgd_kernel");
  return AGNN_OK;
}
