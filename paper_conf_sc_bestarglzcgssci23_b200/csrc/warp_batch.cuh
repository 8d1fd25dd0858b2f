// warp_batch.cuh — helpers shared by the lane-parallel k = 128 sparse kernels
// (gat_k128.cu, av_k128.cu): the static work-list item of a warp and the
// transposed butterfly reduction that turns B per-lane partial dot products
// into one full dot product per lane.
#pragma once
#include "internal.cuh"

namespace agnn {
namespace wb {

constexpr unsigned FULL = 0xffffffffu;

__device__ __forceinline__ void item_of(const Items& it, int64_t w, int64_t& row, int64_t& beg,
                                        int64_t& end, int64_t& slot) {
  if (w < it.n_chunks) {
    row = it.chunk_row[w];
    beg = it.row_ptr[row] + (int64_t)it.chunk_idx[w] * it.chunk;
    end = min(beg + (int64_t)it.chunk, it.row_ptr[row + 1]);
    slot = w;
  } else {
    row = it.light_rows[w - it.n_chunks];
    beg = it.row_ptr[row];
    end = it.row_ptr[row + 1];
    slot = -1;
  }
}


// Transposed reduction of B partial sums held by every lane of a group of HL lanes:
// afterwards lane-in-group ql holds in x[0] the full sum of element edge_of(ql)
// (T = log2 B exchange steps of halving width, then plain butterflies).
template <int B>
struct Transpose {
  static constexpr int T = (B >= 32) ? 5 : (B >= 16) ? 4 : (B >= 8) ? 3 : (B >= 4) ? 2 : (B >= 2) ? 1 : 0;
  // edge index held by lane-in-group ql after the transposed reduction
  __device__ static __forceinline__ int edge_of(int ql) {
    int b = 0;
#pragma unroll
    for (int s = 0; s < T; ++s) b |= ((ql >> s) & 1) * (B >> (s + 1));
    return b;
  }
  // lane-in-group that holds edge b
  __device__ static __forceinline__ int lane_of(int b) {
    int q = 0;
#pragma unroll
    for (int s = 0; s < T; ++s) q |= ((b / (B >> (s + 1))) & 1) << s;
    return q;
  }
  // x[0..B) partial sums over the HL lanes of a head group -> x[0] = full sum of
  // element edge_of(lane % HL), every lane
  template <int HL>
  __device__ static __forceinline__ void reduce(float (&x)[B], int lane) {
    int len = B;
#pragma unroll
    for (int s = 0; s < T; ++s) {
      const int o = 1 << s;
      const bool upper = (lane & o) != 0;
      len >>= 1;
#pragma unroll
      for (int k = 0; k < B / 2; ++k) {
        if (k < len) {
          const float keep = upper ? x[k + len] : x[k];
          const float send = upper ? x[k] : x[k + len];
          x[k] = keep + __shfl_xor_sync(wb::FULL, send, o);
        }
      }
    }
#pragma unroll
    for (int o = B; o < HL; o <<= 1) x[0] += __shfl_xor_sync(wb::FULL, x[0], o);
  }
};


}  // namespace wb
}  // namespace agnn
