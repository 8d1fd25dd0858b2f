// csr_build.cu — agnn_csr_build: the paper's graph preprocessing on the device.
//
// PAPER.md:574 (artifact): Kronecker graphs are generated, duplicates removed
// and every vertex connected to at least one other vertex; PAPER.md:75 uses
// N^(v) = N(v) u {v}.  Readings A1-A3/A21: drop self-pairs,
// (optionally) symmetrise, dedup, connect every vertex without a non-self
// neighbour to (v+1) mod n in both directions, add (v,v) for every v; rows
// ascending, columns strictly ascending.  Radix sort + unique on 64-bit keys
// (row << 32 | col) with CUB.  Utility, not on the timed path; synchronises.
#include <cub/cub.cuh>

#include "internal.cuh"

namespace agnn {
namespace {

__global__ void make_keys_kernel(const uint32_t* __restrict__ src, const uint32_t* __restrict__ dst,
                                 int64_t n_pairs, int sym, uint64_t sentinel,
                                 uint64_t* __restrict__ keys) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n_pairs;
       e += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t s = src[e], d = dst[e];
    const bool self = s == d;
    keys[sym ? 2 * e : e] = self ? sentinel : ((s << 32) | d);
    if (sym) keys[2 * e + 1] = self ? sentinel : ((d << 32) | s);
  }
}

__global__ void range_check_kernel(const uint32_t* __restrict__ src,
                                   const uint32_t* __restrict__ dst, int64_t n_pairs, int64_t n,
                                   int* __restrict__ bad) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n_pairs;
       e += (int64_t)gridDim.x * blockDim.x)
    if ((int64_t)src[e] >= n || (int64_t)dst[e] >= n) *bad = 1;
}

// row_ptr[v] = first position p with (keys[p] >> 32) >= v   (keys sorted)
__global__ void row_ptr_kernel(const uint64_t* __restrict__ keys, int64_t cnt, int64_t n,
                               int64_t* __restrict__ rp) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v <= n;
       v += (int64_t)gridDim.x * blockDim.x) {
    int64_t lo = 0, hi = cnt;
    const uint64_t key = (uint64_t)v << 32;
    while (lo < hi) {
      const int64_t mid = lo + (hi - lo) / 2;
      if (keys[mid] < key) lo = mid + 1; else hi = mid;
    }
    rp[v] = lo;
  }
}

// extra keys: self-loops for all v, and the A2 connection for vertices without neighbours
__global__ void extra_keys_kernel(const int64_t* __restrict__ rp, int64_t n, int self_loops,
                                  int connect, uint64_t* __restrict__ out, uint64_t sentinel) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    uint64_t* o = out + 3 * v;
    o[0] = self_loops ? (((uint64_t)v << 32) | (uint64_t)v) : sentinel;
    const bool iso = connect && n > 1 && rp[v + 1] == rp[v];
    const uint64_t u = (uint64_t)((v + 1) % n);
    o[1] = iso ? (((uint64_t)v << 32) | u) : sentinel;
    o[2] = iso ? ((u << 32) | (uint64_t)v) : sentinel;
  }
}

__global__ void low_bits_kernel(const uint64_t* __restrict__ keys, int64_t cnt,
                                int32_t* __restrict__ col) {
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < cnt;
       p += (int64_t)gridDim.x * blockDim.x)
    col[p] = (int32_t)(keys[p] & 0xFFFFFFFFull);
}

int bits_for(int64_t n) {
  int b = 1;
  while (((int64_t)1 << b) <= n) ++b;
  return b;
}

// CSC keys (col << 32 | row) and CSR positions of every stored entry (warp per row)
__global__ void csc_keys_kernel(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                int64_t n_rows, uint64_t* __restrict__ keys,
                                int64_t* __restrict__ pos) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n_rows; i += nw) {
    for (int64_t e = rp[i] + lane; e < rp[i + 1]; e += 32) {
      keys[e] = ((uint64_t)(uint32_t)col[e] << 32) | (uint64_t)i;
      if (pos) pos[e] = e;
    }
  }
}

}  // namespace

// CSC of a local CSR (rows [0, n_rows), global columns < n): entries sorted by
// (column, row); csc_ptr[j] = first entry of column j; perm[e_csc] = CSR position.
// Plan-time utility (radix sort on the device; synchronises).
agnn_status build_csc(const int64_t* row_ptr, const int32_t* col, int64_t n_rows, int64_t n,
                      int64_t nnz, int64_t* csc_ptr, int32_t* csc_idx, int64_t* perm,
                      cudaStream_t s) {
  const int grid = kNumSMs * 8;
  if (nnz == 0) {
    AGNN_CUDA_TRY(cudaMemsetAsync(csc_ptr, 0, sizeof(int64_t) * (size_t)(n + 1), s));
    AGNN_CUDA_TRY(cudaStreamSynchronize(s));
    return AGNN_OK;
  }
  uint64_t *ka = nullptr, *kb = nullptr;
  int64_t *va = nullptr, *vb = nullptr;
  void* tmp = nullptr;
  agnn_status st = AGNN_OK;
  auto cleanup = [&]() {
    if (ka) cudaFreeAsync(ka, s);
    if (kb) cudaFreeAsync(kb, s);
    if (va) cudaFreeAsync(va, s);
    if (vb) cudaFreeAsync(vb, s);
    if (tmp) cudaFreeAsync(tmp, s);
    cudaStreamSynchronize(s);
  };
  do {
    if ((st = cuda_status(cudaMallocAsync(&ka, sizeof(uint64_t) * nnz, s), "csc malloc")) != AGNN_OK) break;
    if ((st = cuda_status(cudaMallocAsync(&kb, sizeof(uint64_t) * nnz, s), "csc malloc")) != AGNN_OK) break;
    if (perm) {
      if ((st = cuda_status(cudaMallocAsync(&va, sizeof(int64_t) * nnz, s), "csc malloc")) != AGNN_OK) break;
      if ((st = cuda_status(cudaMallocAsync(&vb, sizeof(int64_t) * nnz, s), "csc malloc")) != AGNN_OK) break;
    }
    csc_keys_kernel<<<grid, 256, 0, s>>>(row_ptr, col, n_rows, ka, va);
    count_launch();
    const int end_bit = 32 + bits_for(n);
    size_t need = 0;
    cub::DoubleBuffer<uint64_t> dk(ka, kb);
    cub::DoubleBuffer<int64_t> dv(va, vb);
    if (perm) st = cuda_status(cub::DeviceRadixSort::SortPairs(nullptr, need, dk, dv, nnz, 0, end_bit, s), "csc sort");
    else st = cuda_status(cub::DeviceRadixSort::SortKeys(nullptr, need, dk, nnz, 0, end_bit, s), "csc sort");
    if (st != AGNN_OK) break;
    if ((st = cuda_status(cudaMallocAsync(&tmp, need, s), "csc malloc")) != AGNN_OK) break;
    if (perm) st = cuda_status(cub::DeviceRadixSort::SortPairs(tmp, need, dk, dv, nnz, 0, end_bit, s), "csc sort");
    else st = cuda_status(cub::DeviceRadixSort::SortKeys(tmp, need, dk, nnz, 0, end_bit, s), "csc sort");
    if (st != AGNN_OK) break;
    count_launch(4);
    row_ptr_kernel<<<grid, 256, 0, s>>>(dk.Current(), nnz, n, csc_ptr);
    low_bits_kernel<<<grid, 256, 0, s>>>(dk.Current(), nnz, csc_idx);
    count_launch(2);
    if (perm)
      st = cuda_status(cudaMemcpyAsync(perm, dv.Current(), sizeof(int64_t) * nnz,
                                       cudaMemcpyDeviceToDevice, s), "csc perm copy");
    if (st == AGNN_OK) st = cuda_status(cudaGetLastError(), "csc kernels");
  } while (0);
  cleanup();
  return st;
}

namespace {
}  // namespace
}  // namespace agnn

using namespace agnn;

// sort keys[0..cnt) (double-buffered), unique into the other buffer; returns count
static agnn_status sort_unique(uint64_t*& a, uint64_t*& b, int64_t cnt, int end_bit, void*& tmp,
                               size_t& tmp_bytes, int64_t* d_cnt, int64_t& out_cnt,
                               cudaStream_t s) {
  cub::DoubleBuffer<uint64_t> db(a, b);
  size_t need = 0;
  AGNN_CUDA_TRY(cub::DeviceRadixSort::SortKeys(nullptr, need, db, cnt, 0, end_bit, s));
  size_t need2 = 0;
  AGNN_CUDA_TRY(cub::DeviceSelect::Unique(nullptr, need2, a, b, d_cnt, cnt, s));
  need = std::max(need, need2);
  if (need > tmp_bytes) {
    if (tmp) AGNN_CUDA_TRY(cudaFreeAsync(tmp, s));
    AGNN_CUDA_TRY(cudaMallocAsync(&tmp, need, s));
    tmp_bytes = need;
  }
  AGNN_CUDA_TRY(cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, db, cnt, 0, end_bit, s));
  count_launch(4);
  uint64_t* sorted = db.Current();
  uint64_t* other = db.Alternate();
  AGNN_CUDA_TRY(cub::DeviceSelect::Unique(tmp, tmp_bytes, sorted, other, d_cnt, cnt, s));
  count_launch(2);
  AGNN_CUDA_TRY(cudaMemcpyAsync(&out_cnt, d_cnt, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
  AGNN_CUDA_TRY(cudaStreamSynchronize(s));
  a = other;   // unique output
  b = sorted;  // free buffer
  return AGNN_OK;
}

extern "C" agnn_status agnn_csr_build(int64_t n, const uint32_t* src, const uint32_t* dst,
                                      int64_t n_pairs, uint32_t flags, int64_t* row_ptr,
                                      int32_t** col_idx, int64_t* nnz_out, cudaStream_t s) {
  if (n <= 0 || n > INT32_MAX || n_pairs < 0 || !row_ptr || !col_idx || !nnz_out ||
      (n_pairs > 0 && (!src || !dst)))
    return fail(AGNN_EINVAL, "agnn_csr_build: bad arguments");
  const int sym = (flags & AGNN_BUILD_SYMMETRIZE) ? 1 : 0;
  const uint64_t sentinel = (uint64_t)n << 32;   // sorts after every real key
  const int end_bit = 32 + bits_for(n);
  const int64_t cap = (sym ? 2 : 1) * n_pairs + 3 * n;
  uint64_t *ka = nullptr, *kb = nullptr;
  int64_t* d_cnt = nullptr;
  int* d_bad = nullptr;
  void* tmp = nullptr;
  size_t tmp_bytes = 0;
  agnn_status st = AGNN_OK;
  int64_t cnt = 0;
  const int grid = kNumSMs * 8;
  auto cleanup = [&]() {
    if (ka) cudaFreeAsync(ka, s);
    if (kb) cudaFreeAsync(kb, s);
    if (d_cnt) cudaFreeAsync(d_cnt, s);
    if (d_bad) cudaFreeAsync(d_bad, s);
    if (tmp) cudaFreeAsync(tmp, s);
    cudaStreamSynchronize(s);
  };
#define TRY(x)                 \
  do {                         \
    st = (x);                  \
    if (st != AGNN_OK) {       \
      cleanup();               \
      return st;               \
    }                          \
  } while (0)
#define CTRY(x) TRY(cuda_status((x), #x))
  CTRY(cudaMallocAsync(&ka, sizeof(uint64_t) * cap, s));
  CTRY(cudaMallocAsync(&kb, sizeof(uint64_t) * cap, s));
  CTRY(cudaMallocAsync(&d_cnt, sizeof(int64_t), s));
  CTRY(cudaMallocAsync(&d_bad, sizeof(int), s));
  CTRY(cudaMemsetAsync(d_bad, 0, sizeof(int), s));
  if (n_pairs > 0) {
    range_check_kernel<<<grid, 256, 0, s>>>(src, dst, n_pairs, n, d_bad);
    make_keys_kernel<<<grid, 256, 0, s>>>(src, dst, n_pairs, sym, sentinel, ka);
    count_launch(2);
    CTRY(cudaGetLastError());
  }
  int h_bad = 0;
  CTRY(cudaMemcpyAsync(&h_bad, d_bad, sizeof(int), cudaMemcpyDeviceToHost, s));
  CTRY(cudaStreamSynchronize(s));
  if (h_bad) {
    cleanup();
    return fail(AGNN_EINVAL, "agnn_csr_build: vertex id out of range");
  }
  cnt = (sym ? 2 : 1) * n_pairs;
  if (cnt > 0) TRY(sort_unique(ka, kb, cnt, end_bit, tmp, tmp_bytes, d_cnt, cnt, s));
  if (cnt > 0) {  // drop the sentinel (self-pairs), which sorts last
    uint64_t last = 0;
    CTRY(cudaMemcpyAsync(&last, ka + cnt - 1, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    CTRY(cudaStreamSynchronize(s));
    if (last == sentinel) --cnt;
  }
  if (flags & (AGNN_BUILD_SELF_LOOPS | AGNN_BUILD_CONNECT_ISOLATED)) {
    row_ptr_kernel<<<grid, 256, 0, s>>>(ka, cnt, n, row_ptr);
    extra_keys_kernel<<<grid, 256, 0, s>>>(row_ptr, n, (flags & AGNN_BUILD_SELF_LOOPS) ? 1 : 0,
                                           (flags & AGNN_BUILD_CONNECT_ISOLATED) ? 1 : 0, ka + cnt,
                                           sentinel);
    count_launch(2);
    CTRY(cudaGetLastError());
    cnt += 3 * n;
    TRY(sort_unique(ka, kb, cnt, end_bit, tmp, tmp_bytes, d_cnt, cnt, s));
    uint64_t last = 0;
    CTRY(cudaMemcpyAsync(&last, ka + cnt - 1, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    CTRY(cudaStreamSynchronize(s));
    if (last == sentinel) --cnt;
  }
  row_ptr_kernel<<<grid, 256, 0, s>>>(ka, cnt, n, row_ptr);
  count_launch();
  int32_t* col = nullptr;
  CTRY(cudaMalloc(&col, sizeof(int32_t) * (cnt > 0 ? cnt : 1)));
  low_bits_kernel<<<grid, 256, 0, s>>>(ka, cnt, col);
  count_launch();
  CTRY(cudaGetLastError());
  cleanup();
  *col_idx = col;
  *nnz_out = cnt;
  return AGNN_OK;
#undef TRY
#undef CTRY
}

extern "C" void agnn_free(void* p) {
  if (p) cudaFree(p);
}
