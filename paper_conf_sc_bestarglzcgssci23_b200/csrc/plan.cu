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
#include <cmath>
#include <cstdlib>
#include <mutex>
#include <unordered_map>
#include <vector>

#include "internal.cuh"

namespace agnn {

namespace {

enum : int { ERR_ROWPTR0 = 1, ERR_ROWPTR_MONO = 2, ERR_COL_RANGE = 4, ERR_COL_ORDER = 8,
             ERR_ASYMMETRIC = 16 };

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

// AGNN_PLAN_VERIFY_SYMMETRY ("for undirected graphs A = A^T"): every
// stored (i,j) must have (j,i) stored — a binary search for i in row j, one lane per
// entry.  Needs every row (world == 1) and a CSR that passed validate_kernel.
__global__ void symmetry_kernel(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                int64_t n, int* __restrict__ err) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < n; i += nw) {
    bool bad = false;
    for (int64_t p = rp[i] + lane; p < rp[i + 1]; p += 32) {
      const int64_t j = col[p];
      int64_t lo = rp[j], hi = rp[j + 1];
      while (lo < hi) {  // first position in row j with column >= i
        const int64_t mid = lo + (hi - lo) / 2;
        if ((int64_t)col[mid] < i) lo = mid + 1; else hi = mid;
      }
      bad |= !(lo < rp[j + 1] && (int64_t)col[lo] == i);
    }
    if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(err, ERR_ASYMMETRIC);
  }
}

// occurrences of every column id in the local CSR (how often a pass gathers row j)
__global__ void col_count_kernel(const int32_t* __restrict__ col, int64_t nnz,
                                 int32_t* __restrict__ cnt) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz;
       e += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + col[e], 1);
}

struct ClassThresholds {
  int32_t t[kMaxColClasses];  // t[q], q = 1..nq-1: class >= q iff count >= t[q] (nondecreasing)
  int nq, shift;
};

// col_hint[e] = col[e] | class(col[e]) << shift
__global__ void col_class_kernel(const int32_t* __restrict__ col, int64_t nnz,
                                 const int32_t* __restrict__ cnt, ClassThresholds th,
                                 int32_t* __restrict__ out) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = col[e], k = cnt[c];
    int q = 0;
    while (q + 1 < th.nq && k >= th.t[q + 1]) ++q;
    out[e] = (int32_t)((uint32_t)c | ((uint32_t)q << th.shift));
  }
}

// Column classes for the L2 residency hints.  Class >= q (q = 1, 2, ...) = the
// column is among the R_q = 2^21 / 2^((q-1)/4) vertices this rank gathers most
// often (ties at a threshold are all left out; a vertex gathered once is never
// hot).  The classes sit in the free high bits of the column ids.  Plan time
// only; synchronises.
agnn_status build_col_classes(Plan& p, cudaStream_t s) {
  int shift = 1;
  while (((int64_t)1 << shift) < p.n) ++shift;
  const int nq = std::min(kMaxColClasses, 1 << std::max(0, 31 - shift));
  if (p.nnz == 0 || p.l2_hot_mb <= 0 || nq < 2) return AGNN_OK;
  int32_t* cnt = nullptr;
  AGNN_CUDA_TRY(cudaMallocAsync(&cnt, sizeof(int32_t) * (size_t)p.n, s));
  AGNN_CUDA_TRY(cudaMemsetAsync(cnt, 0, sizeof(int32_t) * (size_t)p.n, s));
  col_count_kernel<<<kNumSMs * 8, 256, 0, s>>>(p.col_idx, p.nnz, cnt);
  AGNN_LAUNCH_CHECK("col_count_kernel");
  std::vector<int32_t> hc((size_t)p.n);
  AGNN_CUDA_TRY(cudaMemcpyAsync(hc.data(), cnt, sizeof(int32_t) * hc.size(),
                                cudaMemcpyDeviceToHost, s));
  AGNN_CUDA_TRY(cudaStreamSynchronize(s));
  int32_t maxc = 0;
  for (int32_t c : hc) maxc = std::max(maxc, c);
  std::vector<int64_t> ge((size_t)maxc + 2, 0);  // ge[t] = #{count >= t}
  for (int32_t c : hc) ++ge[(size_t)c];
  for (int64_t t = maxc - 1; t >= 0; --t) ge[(size_t)t] += ge[(size_t)t + 1];
  ClassThresholds th;
  th.nq = nq;
  th.shift = shift;
  th.t[0] = 0;
  p.class_rows[0] = p.n;
  int64_t t = 2;
  for (int q = 1; q < nq; ++q) {
    const double R = std::ldexp(1.0, 21) / std::pow(2.0, (q - 1) / 4.0);
    while (t <= maxc && (double)ge[(size_t)t] > R) ++t;
    th.t[q] = (int32_t)std::min<int64_t>(t, (int64_t)maxc + 1);
    p.class_rows[q] = th.t[q] <= maxc ? ge[(size_t)th.t[q]] : 0;
  }
  p.hint_shift = shift;
  p.n_classes = nq;
  AGNN_CUDA_TRY(cudaMalloc(&p.col_hint, sizeof(int32_t) * (size_t)p.nnz));
  col_class_kernel<<<kNumSMs * 8, 256, 0, s>>>(p.col_idx, p.nnz, cnt, th, p.col_hint);
  AGNN_LAUNCH_CHECK("col_class_kernel");
  AGNN_CUDA_TRY(cudaFreeAsync(cnt, s));
  AGNN_CUDA_TRY(cudaStreamSynchronize(s));
  return AGNN_OK;
}

}  // namespace

// every gathered row outside the hot set is loaded evict_first (measured C5, round 1:
// evict_last alone, without evict_first for the rest, gave nothing)
Items l2_hinted(const Items& it, const Plan& p, int64_t row_bytes) {
  if (!p.col_hint || it.col != p.col_idx || row_bytes <= 0) return it;
  const int64_t budget = p.l2_hot_mb << 20;
  int q = 1;
  while (q < p.n_classes && p.class_rows[q] * row_bytes > budget) ++q;
  Items r = it;
  r.col = p.col_hint;
  r.col_mask = (1u << p.hint_shift) - 1u;
  r.hot_thr = q < p.n_classes ? (uint32_t)q << p.hint_shift : 0xffffffffu;
  r.cold_first = 1;
  return r;
}

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
  it.short_rows = p.short_rows;
  it.short_meta = p.short_meta;
  it.n_short = p.n_short;
  it.n_short_nz = p.n_short_nz;
  it.bundles = p.bundles;
  it.n_bundles = p.n_bundles;
  it.long_rows = p.long_rows;
  it.n_long = p.n_long;
  it.bundle_mode = p.bundle_mode;
  return it;
}

namespace {

// static work list of one pattern (rows of the CSR, or columns of the CSC)
struct Lists {
  int64_t n_light = 0, n_heavy = 0, n_chunks = 0, n_empty = 0, max_deg = 0, n_short = 0,
          n_long = 0;
  int32_t *light = nullptr, *chunk_row = nullptr, *chunk_idx = nullptr, *heavy = nullptr,
          *heavy_off = nullptr, *empty = nullptr, *short_rows = nullptr, *long_rows = nullptr;
  void* block = nullptr;
};

agnn_status build_lists(const std::vector<int64_t>& rp, int64_t n_rows, int chunk, bool with_empty,
                        int short_max, Lists& out, cudaStream_t s) {
  std::vector<int32_t> light, chunk_row, chunk_idx, heavy, heavy_off{0}, empty, shorts, longs;
  light.reserve((size_t)n_rows);
  int64_t maxdeg = 0;
  for (int64_t i = 0; i < n_rows; ++i) {
    const int64_t d = rp[(size_t)i + 1] - rp[(size_t)i];
    maxdeg = std::max(maxdeg, d);
    if (d == 0 && with_empty) empty.push_back((int32_t)i);
    if (d > chunk) {
      const int64_t c = (d + chunk - 1) / chunk;
      heavy.push_back((int32_t)i);
      for (int64_t q = 0; q < c; ++q) {
        chunk_row.push_back((int32_t)i);
        chunk_idx.push_back((int32_t)q);
      }
      heavy_off.push_back((int32_t)chunk_row.size());
    } else {
      light.push_back((int32_t)i);
      if (short_max > 0) (d <= short_max ? shorts : longs).push_back((int32_t)i);
    }
  }
  out.max_deg = maxdeg;
  out.n_light = (int64_t)light.size();
  out.n_heavy = (int64_t)heavy.size();
  out.n_chunks = (int64_t)chunk_row.size();
  out.n_empty = (int64_t)empty.size();
  out.n_short = (int64_t)shorts.size();
  out.n_long = (int64_t)longs.size();
  const size_t total = light.size() + 2 * chunk_row.size() + heavy.size() + heavy_off.size() +
                       empty.size() + shorts.size() + longs.size() + 160;
  AGNN_CUDA_TRY(cudaMalloc(&out.block, sizeof(int32_t) * total));
  int32_t* b = static_cast<int32_t*>(out.block);
  auto put = [&](std::vector<int32_t>& v, int32_t*& dst) -> cudaError_t {
    dst = b;
    b += v.size() + 16 - (v.size() % 16);
    if (v.empty()) return cudaSuccess;
    return cudaMemcpyAsync(dst, v.data(), sizeof(int32_t) * v.size(), cudaMemcpyHostToDevice, s);
  };
  AGNN_CUDA_TRY(put(light, out.light));
  AGNN_CUDA_TRY(put(chunk_row, out.chunk_row));
  AGNN_CUDA_TRY(put(chunk_idx, out.chunk_idx));
  AGNN_CUDA_TRY(put(heavy, out.heavy));
  AGNN_CUDA_TRY(put(heavy_off, out.heavy_off));
  AGNN_CUDA_TRY(put(empty, out.empty));
  AGNN_CUDA_TRY(put(shorts, out.short_rows));
  AGNN_CUDA_TRY(put(longs, out.long_rows));
  AGNN_CUDA_TRY(cudaStreamSynchronize(s));  // the host vectors die here
  return AGNN_OK;
}

}  // namespace

Items items_of_csc(const Plan& p) {
  Items it;
  it.row_ptr = p.csc_ptr;
  it.col = p.csc_idx;
  it.light_rows = p.c_light_rows;
  it.n_light = p.c_light;
  it.chunk_row = p.c_chunk_row;
  it.chunk_idx = p.c_chunk_idx;
  it.n_chunks = p.c_chunks;
  it.chunk = p.chunk;
  it.heavy_rows = p.c_heavy_rows;
  it.heavy_off = p.c_heavy_off;
  it.n_heavy = p.c_heavy;
  it.row_begin = 0;
  it.n_local = p.n;
  it.short_rows = it.long_rows = nullptr;
  it.short_meta = nullptr;
  it.bundles = nullptr;
  it.n_bundles = it.n_short_nz = 0;
  it.n_short = it.n_long = 0;
  return it;
}

// heavy-row chunk size (edges): the longest item bounds a launch, so smaller graphs
// (fewer edges per resident warp) take smaller chunks.  A function of the GLOBAL n
// only, so chunk boundaries, and with them the summation order, are the same for
// every number of GPUs: 256 up to n = 2^21, doubling per doubling of n, <= 2048
// (measured: C2 1.49e9 -> 2.72e9 edges/s, C3 +11 %, C4 +8 %, C5 unchanged).
// Options (agnn_plan_options): tests take small chunks to exercise the split/merge
// path on small graphs; short rows (degree <= short_max, a function of the degree
// only, like the chunks) go to the short-row kernels where a kernel has one.
agnn_status plan_options(Plan& p, const agnn_plan_options* o) {
  int64_t c = 256;
  for (int64_t t = (int64_t)1 << 21; t < p.n && c < 2048; t <<= 1) c <<= 1;
  p.chunk = (int)c;
  if (!o) return AGNN_OK;
  if (o->chunk_edges != 0) {
    if (o->chunk_edges < 32 || o->chunk_edges > (1 << 30))
      return fail(AGNN_EINVAL, "agnn_plan_options: chunk_edges must be 0 or in 32 .. 2^30");
    p.chunk = o->chunk_edges;
  }
  if (o->short_edges >= 0) {
    if (o->short_edges > 32) return fail(AGNN_EINVAL, "agnn_plan_options: short_edges > 32");
    p.short_max = o->short_edges;
  }
  if (o->short_bundles >= 0) {
    if (o->short_bundles > 2) return fail(AGNN_EINVAL, "agnn_plan_options: short_bundles > 2");
    p.bundle_mode = o->short_bundles;
  }
  if (o->gat_factored >= 0) {
    if (o->gat_factored > 2) return fail(AGNN_EINVAL, "agnn_plan_options: gat_factored > 2");
    p.gat_factored = o->gat_factored;
  }
  if (o->l2_hot_mb >= 0) p.l2_hot_mb = o->l2_hot_mb;
  if (o->spmmm >= 0) {
    if (o->spmmm > 1) return fail(AGNN_EINVAL, "agnn_plan_options: spmmm > 1");
    p.spmmm = o->spmmm;
  }
  return AGNN_OK;
}

agnn_status plan_build(Plan& p, cudaStream_t s) {
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
  if (p.flags & AGNN_PLAN_VERIFY_SYMMETRY) {
    if (p.world != 1 || p.n_local != p.n)
      return fail(AGNN_EUNSUPPORTED,
                  "agnn_plan_create: AGNN_PLAN_VERIFY_SYMMETRY needs world == 1 (every row)");
    int* d_sym = nullptr;
    AGNN_CUDA_TRY(cudaMallocAsync(&d_sym, sizeof(int), s));
    AGNN_CUDA_TRY(cudaMemsetAsync(d_sym, 0, sizeof(int), s));
    if (p.nnz > 0) {
      symmetry_kernel<<<kNumSMs * 8, 256, 0, s>>>(p.row_ptr, p.col_idx, p.n, d_sym);
      AGNN_LAUNCH_CHECK("symmetry_kernel");
    }
    int h_sym = 0;
    AGNN_CUDA_TRY(cudaMemcpyAsync(&h_sym, d_sym, sizeof(int), cudaMemcpyDeviceToHost, s));
    AGNN_CUDA_TRY(cudaStreamSynchronize(s));
    AGNN_CUDA_TRY(cudaFreeAsync(d_sym, s));
    if (h_sym)
      return fail(AGNN_EINVAL,
                  "agnn_plan_create: AGNN_PLAN_VERIFY_SYMMETRY: the pattern is not symmetric "
                  "(a stored (i,j) has no stored (j,i))");
  }
  // 3. work lists of the rows
  Lists L;
  agnn_status st = build_lists(rp, p.n_local, p.chunk, true, p.short_max, L, s);
  if (st != AGNN_OK) return st;
  p.max_deg = L.max_deg;
  p.n_light = L.n_light;
  p.n_heavy = L.n_heavy;
  p.n_chunks = L.n_chunks;
  p.n_empty = L.n_empty;
  p.light_rows = L.light;
  p.chunk_row = L.chunk_row;
  p.chunk_idx = L.chunk_idx;
  p.heavy_rows = L.heavy;
  p.heavy_off = L.heavy_off;
  p.empty_rows = L.empty;
  p.n_short = L.n_short;
  p.n_long = L.n_long;
  p.short_rows = L.short_rows;
  p.long_rows = L.long_rows;
  if (p.n_short > 0) {
    // {row, degree, beg} of every short row in one 16-byte record (the short-row
    // kernels prefetch the next rows' records and column ids a step ahead)
    std::vector<int4> meta;
    std::vector<int32_t> srows((size_t)p.n_short);
    AGNN_CUDA_TRY(cudaMemcpyAsync(srows.data(), p.short_rows, sizeof(int32_t) * srows.size(),
                                  cudaMemcpyDeviceToHost, s));
    AGNN_CUDA_TRY(cudaStreamSynchronize(s));
    // rows with stored entries first (ascending), then the empty rows: the bundles
    // below cover exactly the first n_short_nz records
    meta.reserve(srows.size());
    for (int pass = 0; pass < 2; ++pass)
      for (size_t x = 0; x < srows.size(); ++x) {
        const int64_t r = srows[x], b = rp[(size_t)r], d = rp[(size_t)r + 1] - b;
        if ((d > 0) != (pass == 0)) continue;
        meta.push_back(make_int4(srows[x], (int)d, (int)(uint32_t)(uint64_t)b,
                                 (int)(uint32_t)((uint64_t)b >> 32)));
      }
    p.n_short_nz = 0;
    while (p.n_short_nz < (int64_t)meta.size() && meta[(size_t)p.n_short_nz].y > 0) ++p.n_short_nz;
    // bundles: consecutive non-empty short rows packed greedily into groups of at most
    // kBundleEdges stored entries, {first record, rows, entries, 0}; a warp takes one
    // bundle as one batch (the bundle kernels, gat_short.cu)
    std::vector<int4> bund;
    for (int64_t x = 0; x < p.n_short_nz;) {
      int64_t e = 0, y = x;
      while (y < p.n_short_nz && e + meta[(size_t)y].y <= kBundleEdges) e += meta[(size_t)y++].y;
      bund.push_back(make_int4((int)x, (int)(y - x), (int)e, 0));
      x = y;
    }
    p.n_bundles = (int64_t)bund.size();
    AGNN_CUDA_TRY(cudaMalloc(&p.short_block, sizeof(int4) * (meta.size() + bund.size())));
    p.short_meta = static_cast<int4*>(p.short_block);
    p.bundles = p.short_meta + meta.size();
    AGNN_CUDA_TRY(cudaMemcpyAsync(p.short_meta, meta.data(), sizeof(int4) * meta.size(),
                                  cudaMemcpyHostToDevice, s));
    if (!bund.empty())
      AGNN_CUDA_TRY(cudaMemcpyAsync(p.bundles, bund.data(), sizeof(int4) * bund.size(),
                                    cudaMemcpyHostToDevice, s));
    AGNN_CUDA_TRY(cudaStreamSynchronize(s));
  }
  p.meta_block = L.block;
  // L2 residency classes of the columns (symmetric or directed; the row pass's gathers)
  if ((st = build_col_classes(p, s)) != AGNN_OK) return st;
  // 4. directed pattern on one GPU: the CSC and its work lists (column role of the backward)
  if (p.directed() && p.world == 1 && p.n_local == p.n) {
    const size_t ptr_bytes = ((sizeof(int64_t) * (size_t)(p.n + 1)) + 255) & ~size_t(255);
    AGNN_CUDA_TRY(cudaMalloc(&p.csc_block, ptr_bytes + sizeof(int32_t) * (size_t)(p.nnz + 1)));
    p.csc_ptr = static_cast<int64_t*>(p.csc_block);
    p.csc_idx = reinterpret_cast<int32_t*>(static_cast<char*>(p.csc_block) + ptr_bytes);
    if ((st = build_csc(p.row_ptr, p.col_idx, p.n_local, p.n, p.nnz, p.csc_ptr, p.csc_idx, nullptr,
                        s)) != AGNN_OK)
      return st;
    std::vector<int64_t> cp((size_t)p.n + 1);
    AGNN_CUDA_TRY(cudaMemcpyAsync(cp.data(), p.csc_ptr, sizeof(int64_t) * cp.size(),
                                  cudaMemcpyDeviceToHost, s));
    AGNN_CUDA_TRY(cudaStreamSynchronize(s));
    Lists C;
    if ((st = build_lists(cp, p.n, p.chunk, false, 0, C, s)) != AGNN_OK) return st;
    p.c_light = C.n_light;
    p.c_heavy = C.n_heavy;
    p.c_chunks = C.n_chunks;
    p.c_light_rows = C.light;
    p.c_chunk_row = C.chunk_row;
    p.c_chunk_idx = C.chunk_idx;
    p.c_heavy_rows = C.heavy;
    p.c_heavy_off = C.heavy_off;
    p.c_meta_block = C.block;
  }
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
