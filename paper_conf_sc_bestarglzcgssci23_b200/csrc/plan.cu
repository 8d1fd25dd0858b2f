// plan.cu — CSR validation, work lists and the 1D partition (agnn_plan_create).
//
// The plan is the only stateful object: it validates the caller's CSR once on
// the device (the one synchronising call, agnn.h "Errors"), and builds the
// static work list used by every sparse kernel:
//   heavy rows (degree > chunk) are split into ceil(deg/chunk) contiguous
//   chunks whose partial results are folded in ascending chunk order;
//   light rows are whole items.  Heavy chunks come first in the list.
// Chunk boundaries depend only on the row degree, so results are identical for
// any launch geometry and any number of GPUs (the row is always computed by its
// owner in the same order).
#include <algorithm>
#include <cstdlib>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "internal.cuh"

namespace agnn {

namespace {

enum : int { ERR_ROWPTR0 = 1, ERR_ROWPTR_MONO = 2, ERR_COL_RANGE = 4, ERR_COL_ORDER = 8 };

__global__ void validate_kernel(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                int64_t n_local, int64_t n, int* __restrict__ err) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  if (blockIdx.x == 0 && threadIdx.x == 0 && rp[0] != 0) atomicOr(err, ERR_ROWPTR0);
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n_local; i += nw) {
    const int64_t b = rp[i], e = rp[i + 1];
    if (e < b) {
      if (lane == 0) atomicOr(err, ERR_ROWPTR_MONO);
      continue;
    }
    int bad = 0;
    for (int64_t p = b + lane; p < e; p += 32) {
      const int32_t c = col[p];
      if (c < 0 || (int64_t)c >= n) bad |= ERR_COL_RANGE;
      if (p + 1 < e && col[p + 1] <= c) bad |= ERR_COL_ORDER;
    }
    bad = __reduce_or_sync(0xffffffffu, bad);
    if (bad && lane == 0) atomicOr(err, bad);
  }
}

}  // namespace

int persistent_blocks(const void* func) {
  static std::mutex mu;
  static std::unordered_map<const void*, int> cache;
  std::lock_guard<std::mutex> lock(mu);
  auto itr = cache.find(func);
  if (itr != cache.end()) return itr->second;
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, func, kSparseThreads, 0) != cudaSuccess ||
      per_sm <= 0)
    per_sm = 1;
  int sms = kNumSMs, dev = 0;
  if (cudaGetDevice(&dev) == cudaSuccess)
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int blocks = std::min(sms * per_sm, kMaxSparseBlocks);
  cache[func] = blocks;
  return blocks;
}

Items items_of(const Plan& p) {
  Items it;
  it.row_ptr = p.row_ptr;
  it.col = p.col_idx;
  it.light_rows = p.light_rows;
  it.n_light = p.n_light;
  it.chunk_row = p.chunk_row;
  it.chunk_idx = p.chunk_idx;
  it.n_chunks = p.n_chunks;
  it.chunk = p.chunk;
  it.heavy_rows = p.heavy_rows;
  it.heavy_off = p.heavy_off;
  it.n_heavy = p.n_heavy;
  it.row_begin = p.row_begin;
  it.n_local = p.n_local;
  return it;
}

agnn_status plan_build(Plan& p, cudaStream_t s) {
  // heavy-row chunk size (edges); AGNN_CHUNK_EDGES overrides it (tests use small
  // chunks to exercise the split/merge path on small graphs)
  if (const char* env = getenv("AGNN_CHUNK_EDGES")) {
    const long v = atol(env);
    if (v >= 32 && v <= (1L << 30)) p.chunk = (int)v;
  }
  // 1. validate on the device
  int* d_err = nullptr;
  AGNN_CUDA_TRY(cudaMallocAsync(&d_err, sizeof(int), s));
  AGNN_CUDA_TRY(cudaMemsetAsync(d_err, 0, sizeof(int), s));
  if (p.n_local > 0) {
    validate_kernel<<<kNumSMs * 8, 256, 0, s>>>(p.row_ptr, p.col_idx, p.n_local, p.n, d_err);
    AGNN_LAUNCH_CHECK("validate_kernel");
  }
  // 2. degrees on the host (one copy of row_ptr; plan time only)
  std::vector<int64_t> rp((size_t)p.n_local + 1);
  AGNN_CUDA_TRY(cudaMemcpyAsync(rp.data(), p.row_ptr, sizeof(int64_t) * rp.size(),
                                cudaMemcpyDeviceToHost, s));
  int h_err = 0;
  AGNN_CUDA_TRY(cudaMemcpyAsync(&h_err, d_err, sizeof(int), cudaMemcpyDeviceToHost, s));
  AGNN_CUDA_TRY(cudaStreamSynchronize(s));
  AGNN_CUDA_TRY(cudaFreeAsync(d_err, s));
  if (h_err) {
    std::string m = "agnn_plan_create: invalid CSR:";
    if (h_err & ERR_ROWPTR0) m += " row_ptr[0] != 0;";
    if (h_err & ERR_ROWPTR_MONO) m += " row_ptr not monotone;";
    if (h_err & ERR_COL_RANGE) m += " column id out of [0, n);";
    if (h_err & ERR_COL_ORDER) m += " columns not strictly ascending (unsorted or duplicate);";
    return fail(AGNN_EINVAL, m);
  }
  p.nnz = rp[(size_t)p.n_local];
  // 3. work lists
  std::vector<int32_t> light, chunk_row, chunk_idx, heavy, heavy_off{0}, empty;
  light.reserve((size_t)p.n_local);
  int64_t maxdeg = 0;
  for (int64_t i = 0; i < p.n_local; ++i) {
    const int64_t d = rp[(size_t)i + 1] - rp[(size_t)i];
    maxdeg = std::max(maxdeg, d);
    if (d == 0) empty.push_back((int32_t)i);
    if (d > p.chunk) {
      const int64_t c = (d + p.chunk - 1) / p.chunk;
      heavy.push_back((int32_t)i);
      for (int64_t q = 0; q < c; ++q) {
        chunk_row.push_back((int32_t)i);
        chunk_idx.push_back((int32_t)q);
      }
      heavy_off.push_back((int32_t)chunk_row.size());
    } else {
      light.push_back((int32_t)i);
    }
  }
  p.max_deg = maxdeg;
  p.n_light = (int64_t)light.size();
  p.n_heavy = (int64_t)heavy.size();
  p.n_chunks = (int64_t)chunk_row.size();
  p.n_empty = (int64_t)empty.size();
  const size_t total = light.size() + 2 * chunk_row.size() + heavy.size() + heavy_off.size() +
                       empty.size() + 160;
  AGNN_CUDA_TRY(cudaMalloc(&p.meta_block, sizeof(int32_t) * total));
  int32_t* b = static_cast<int32_t*>(p.meta_block);
  auto put = [&](std::vector<int32_t>& v, int32_t*& dst) -> cudaError_t {
    dst = b;
    b += v.size() + 16 - (v.size() % 16);
    if (v.empty()) return cudaSuccess;
    return cudaMemcpyAsync(dst, v.data(), sizeof(int32_t) * v.size(), cudaMemcpyHostToDevice, s);
  };
  AGNN_CUDA_TRY(put(light, p.light_rows));
  AGNN_CUDA_TRY(put(chunk_row, p.chunk_row));
  AGNN_CUDA_TRY(put(chunk_idx, p.chunk_idx));
  AGNN_CUDA_TRY(put(heavy, p.heavy_rows));
  AGNN_CUDA_TRY(put(heavy_off, p.heavy_off));
  AGNN_CUDA_TRY(put(empty, p.empty_rows));
  AGNN_CUDA_TRY(cudaStreamSynchronize(s));
  return AGNN_OK;
}

}  // namespace agnn

extern "C" agnn_status agnn_partition(int64_t n, const int64_t* rp, int world, int64_t c_v,
                                      int64_t* bounds) {
  if (world < 1 || n < 0 || !bounds || (n > 0 && !rp) || c_v < 0)
    return agnn::fail(AGNN_EINVAL, "agnn_partition: bad arguments");
  // w(r) = row_ptr[r] + c_v r (reading A20); bounds[p] = min{r : w(r) >= ceil(p w(n) / P)}
  const int64_t wn = (n > 0 ? rp[n] : 0) + c_v * n;
  bounds[0] = 0;
  bounds[world] = n;
  for (int p = 1; p < world; ++p) {
    const int64_t target = (p * wn + world - 1) / world;
    int64_t lo = 0, hi = n;  // first r in [0, n] with w(r) >= target (w is monotone)
    while (lo < hi) {
      const int64_t mid = lo + (hi - lo) / 2;
      if (rp[mid] + c_v * mid >= target) hi = mid; else lo = mid + 1;
    }
    bounds[p] = lo;
  }
  return AGNN_OK;
}
