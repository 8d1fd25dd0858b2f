// comm.cu — the multi-GPU exchange steps of the 1D row-block layout.
//
// The paper distributes A-stationary 1.5D/2D blocks over MPI; on
// one NVSwitch box every GPU reaches every peer at full bandwidth, so the build
// uses contiguous row blocks: rank r owns rows [bounds[r], bounds[r+1]) and the
// only exchanges are
//   forward : all-gather of the projected rows (P | s t) or (H | nu)
//   backward: all-gather of G (or M) plus per-vertex records
//             all-reduce of the weight gradients dW, da
// Two transports:
//  * peer memory (default when the caller passes no NCCL id): at setup every
//    rank maps the other ranks' replicated buffers and control block with CUDA
//    IPC (NVLink / NVSwitch loads and stores, agnn_plan_connect /
//    agnn_plan_register).  An all-gather is a kernel that stores rows of this
//    rank's block straight into every peer's replica, fenced by a flag barrier —
//    only the rows the peer's own CSR references (its "wanted" columns in this
//    block, exchanged once at agnn_plan_connect; the GAT projection GEMM epilogue
//    and backward prologue store their rows to the peers themselves by a per-row
//    peer mask, so those exchanges overlap their producers): the sparse kernels gather a
//    replicated row only as the neighbour of a local row, so every row a rank
//    reads arrives and the results are bitwise those of the full all-gather, at
//    ~40-60 % of its NVLink bytes on the Kronecker graphs.  An
//    all-reduce writes this rank's partial into every peer's slot and each rank
//    adds the slots in rank order (identical, deterministic result on every rank).
//  * NCCL: the variable-size all-gather is a group of ncclBroadcast calls (one
//    root per rank, in place), since NCCL has no all-gather-v; ncclAllReduce.
#include <cuda.h>
#include <nccl.h>

#include <algorithm>
#include <map>
#include <mutex>

#include "internal.cuh"

namespace agnn {

namespace {

constexpr int64_t kRedMax = 65536 + 1024;        // floats per rank per reduce slot
constexpr size_t kFlagBytes = 1024;              // int64 flags [kMaxPeers] (padded)

size_t ctl_bytes(int world) { return kFlagBytes + sizeof(float) * 2 * (size_t)world * kRedMax; }
int64_t* flags_of(void* ctl) { return static_cast<int64_t*>(ctl); }
float* red_of(void* ctl, int world, int set, int rank) {
  return reinterpret_cast<float*>(static_cast<char*>(ctl) + kFlagBytes) +
         ((size_t)set * world + rank) * kRedMax;
}

struct PeerPtrs {
  char* p[kMaxPeers];
};
struct PeerOffs {
  int64_t o[kMaxPeers + 1];  // send_off
};

// barrier over the ranks: publish `epoch` into slot [rank] of every peer's flags,
// then wait until every peer has published it into ours (system-scope release /
// acquire, so the data stores issued before by this stream are visible first)
__global__ void peer_barrier_kernel(int64_t* own, PeerPtrs peers, int rank, int world,
                                    int64_t epoch) {
  if (threadIdx.x != 0) return;
  __threadfence_system();
  for (int r = 0; r < world; ++r) {
    if (r == rank) continue;
    int64_t* f = reinterpret_cast<int64_t*>(peers.p[r]) + rank;
    asm volatile("st.release.sys.global.s64 [%0], %1;" ::"l"(f), "l"(epoch) : "memory");
  }
  for (int r = 0; r < world; ++r) {
    if (r == rank) continue;
    int64_t v;
    do {
      asm volatile("ld.acquire.sys.global.s64 %0, [%1];" : "=l"(v) : "l"(own + r) : "memory");
    } while (v < epoch);
  }
}

// the rows of send lists (global row ids, by peer) of the replicated arrays -> the
// same rows of every peer's replica; one warp per (peer, row), every array in turn
struct PushArr {
  const float* src[4];
  PeerPtrs dst[4];
  int64_t width[4];  // floats per row
  int n;
};
__global__ void peer_push_needed_kernel(PushArr A, const int32_t* __restrict__ idx,
                                        int64_t total, PeerOffs offs) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < total; w += nw) {
    int q = 0;
    while (w >= offs.o[q + 1]) ++q;  // peer of list entry w
    const int64_t row = idx[w];
#pragma unroll 1
    for (int a = 0; a < A.n; ++a) {
      const int64_t wd = A.width[a];
      const float* src = A.src[a] + row * wd;
      float* dst = reinterpret_cast<float*>(A.dst[a].p[q]) + row * wd;
      if ((wd & 3) == 0) {
        for (int64_t c = 4 * lane; c < wd; c += 128) st4(dst + c, ldg4(src + c));
      } else {
        for (int64_t c = lane; c < wd; c += 32) dst[c] = src[c];
      }
    }
  }
}

// this rank's partial -> slot [set][rank] of every rank's control block (own included)
__global__ void peer_red_write_kernel(const float* __restrict__ buf, int64_t count, PeerPtrs ctl,
                                      int rank, int world, int set) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
       i += (int64_t)gridDim.x * blockDim.x) {
    const float v = buf[i];
    for (int r = 0; r < world; ++r) {
      float* slot = reinterpret_cast<float*>(ctl.p[r] + kFlagBytes) + ((size_t)set * world + rank) * kRedMax;
      slot[i] = v;
    }
  }
}

// buf[i] = sum over ranks 0..world-1 (fixed order) of the slots
__global__ void peer_red_sum_kernel(const float* __restrict__ slots, int64_t count, int world,
                                    float* __restrict__ buf) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count;
       i += (int64_t)gridDim.x * blockDim.x) {
    float acc = 0.f;
    for (int r = 0; r < world; ++r) acc += slots[(size_t)r * kRedMax + i];
    buf[i] = acc;
  }
}

using PFN_getRange = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
PFN_getRange get_range_fn() {
  static PFN_getRange fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaDriverEntryPointQueryResult q;
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &p, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_getRange>(p);
  });
  return fn;
}

// CUDA IPC maps an allocation at most once per process, while several plans (and
// several registered tensors of one allocation) may need it: the mappings are
// shared and reference-counted.  Every acquisition is recorded in the acquiring
// plan's `opened` list and released by comm_destroy; the mapping is closed when
// its last holder releases it.
struct IpcMap {
  void* base;
  int refs;
};
std::mutex g_ipc_mu;
std::map<std::pair<int, std::string>, IpcMap> g_ipc;

void ipc_release(void* base) {  // caller holds g_ipc_mu
  for (auto it = g_ipc.begin(); it != g_ipc.end(); ++it) {
    if (it->second.base != base) continue;
    if (--it->second.refs == 0) {
      cudaIpcCloseMemHandle(base);
      g_ipc.erase(it);
    }
    return;
  }
}
}  // namespace

// map every peer's IPC handle (rank order, 64 B each) + byte offset; own rank -> local
agnn_status peer_open(Plan& p, const void* handles, const int64_t* offsets, void* local,
                       char* out[kMaxPeers]) {
  std::lock_guard<std::mutex> lock(g_ipc_mu);
  for (int r = 0; r < p.world; ++r) {
    if (r == p.rank) {
      out[r] = static_cast<char*>(local);
      continue;
    }
    cudaIpcMemHandle_t h;
    memcpy(&h, static_cast<const char*>(handles) + 64 * r, sizeof(h));
    const auto key = std::make_pair(r, std::string(reinterpret_cast<const char*>(&h), sizeof(h)));
    void* base = nullptr;
    auto it = g_ipc.find(key);
    if (it != g_ipc.end()) {
      base = it->second.base;
      ++it->second.refs;
    } else {
      AGNN_CUDA_TRY(cudaIpcOpenMemHandle(&base, h, cudaIpcMemLazyEnablePeerAccess));
      g_ipc[key] = IpcMap{base, 1};
    }
    p.opened->push_back(base);
    out[r] = static_cast<char*>(base) + offsets[r];
  }
  return AGNN_OK;
}

namespace {

bool peer_lookup(const Plan& p, const void* addr, PeerPtrs& out) {
  if (!p.regs) return false;
  const char* a = static_cast<const char*>(addr);
  for (const auto& g : *p.regs) {
    if (a >= g.local && a < g.local + g.bytes) {
      for (int r = 0; r < p.world; ++r) out.p[r] = g.peer[r] + (a - g.local);
      return true;
    }
  }
  return false;
}

}  // namespace

agnn_status peer_barrier(const Plan& p, cudaStream_t s) {
  PeerPtrs f;
  for (int r = 0; r < p.world; ++r) f.p[r] = static_cast<char*>(p.peer_ctl[r]);
  peer_barrier_kernel<<<1, 32, 0, s>>>(flags_of(p.ctl), f, p.rank, p.world, ++p.epoch);
  AGNN_LAUNCH_CHECK("peer_barrier_kernel");
  return AGNN_OK;
}

agnn_status peer_targets(const Plan& p, const void* local, void* out[kMaxPeers]) {
  PeerPtrs pp;
  if (!peer_lookup(p, local, pp))
    return fail(AGNN_ESTATE, "peer exchange: buffer not registered (agnn_plan_register)");
  for (int r = 0; r < p.world; ++r) out[r] = pp.p[r];
  return AGNN_OK;
}

__global__ void mark_cols_kernel(const int32_t* __restrict__ col, int64_t nnz,
                                 uint8_t* __restrict__ mark) {
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < nnz;
       e += (int64_t)gridDim.x * blockDim.x)
    mark[col[e]] = 1;
}

// The columns of other ranks' blocks that this rank's CSR references ("wanted"),
// ascending, with per-block offsets, written behind the flags and reduce slots of
// the control block (peers read them at agnn_plan_connect).  Plan time; synchronises.
agnn_status peer_init(Plan& p) {
  p.peer = true;
  p.regs = new std::vector<Plan::Reg>();
  p.opened = new std::vector<void*>();
  std::vector<uint8_t> mark((size_t)p.n, 0);
  if (p.nnz > 0) {
    uint8_t* d_mark = nullptr;
    AGNN_CUDA_TRY(cudaMalloc(&d_mark, (size_t)p.n));
    AGNN_CUDA_TRY(cudaMemset(d_mark, 0, (size_t)p.n));
    mark_cols_kernel<<<kNumSMs * 8, 256>>>(p.col_idx, p.nnz, d_mark);
    AGNN_CUDA_TRY(cudaGetLastError());
    AGNN_CUDA_TRY(cudaMemcpy(mark.data(), d_mark, (size_t)p.n, cudaMemcpyDeviceToHost));
    AGNN_CUDA_TRY(cudaFree(d_mark));
  }
  std::vector<int64_t> woff((size_t)p.world + 1, 0);
  std::vector<int32_t> want;
  for (int q = 0; q < p.world; ++q) {
    woff[(size_t)q] = (int64_t)want.size();
    if (q == p.rank) continue;
    for (int64_t j = p.bounds[q]; j < p.bounds[q + 1]; ++j)
      if (mark[(size_t)j]) want.push_back((int32_t)j);
  }
  woff[(size_t)p.world] = (int64_t)want.size();
  p.n_wanted = (int64_t)want.size();
  p.want_off = (ctl_bytes(p.world) + 255) & ~size_t(255);
  const size_t bytes = p.want_off + sizeof(int64_t) * woff.size() + sizeof(int32_t) * want.size();
  AGNN_CUDA_TRY(cudaMalloc(&p.ctl, bytes));
  AGNN_CUDA_TRY(cudaMemset(p.ctl, 0, ctl_bytes(p.world)));
  char* w = static_cast<char*>(p.ctl) + p.want_off;
  AGNN_CUDA_TRY(cudaMemcpy(w, woff.data(), sizeof(int64_t) * woff.size(), cudaMemcpyHostToDevice));
  if (!want.empty())
    AGNN_CUDA_TRY(cudaMemcpy(w + sizeof(int64_t) * woff.size(), want.data(),
                             sizeof(int32_t) * want.size(), cudaMemcpyHostToDevice));
  AGNN_CUDA_TRY(cudaDeviceSynchronize());
  return AGNN_OK;
}

// agnn_plan_connect: the send lists = every peer's wanted columns in this rank's block
agnn_status peer_send_lists(Plan& p) {
  std::vector<int32_t> all;
  p.send_off[0] = 0;
  for (int q = 0; q < p.world; ++q) {
    if (q != p.rank) {
      const char* w = static_cast<const char*>(p.peer_ctl[q]) + p.want_off;
      int64_t o[2];
      AGNN_CUDA_TRY(cudaMemcpy(o, w + sizeof(int64_t) * p.rank, sizeof(o), cudaMemcpyDeviceToHost));
      const int64_t cnt = o[1] - o[0];
      if (cnt < 0 || cnt > p.n_local)
        return fail(AGNN_ESTATE, "peer exchange: inconsistent wanted lists (plans differ across ranks)");
      const size_t at = all.size();
      all.resize(at + (size_t)cnt);
      if (cnt > 0)
        AGNN_CUDA_TRY(cudaMemcpy(all.data() + at,
                                 w + sizeof(int64_t) * (p.world + 1) + sizeof(int32_t) * o[0],
                                 sizeof(int32_t) * cnt, cudaMemcpyDeviceToHost));
    }
    p.send_off[q + 1] = (int64_t)all.size();
  }
  if (p.send_idx) cudaFree(p.send_idx);
  p.send_idx = nullptr;
  if (!all.empty()) {
    AGNN_CUDA_TRY(cudaMalloc(&p.send_idx, sizeof(int32_t) * all.size()));
    AGNN_CUDA_TRY(cudaMemcpy(p.send_idx, all.data(), sizeof(int32_t) * all.size(),
                             cudaMemcpyHostToDevice));
  }
  // the same lists as a per-row bit mask over the compact peer order (rank order
  // without this rank), for the producing kernels that store the rows themselves
  std::vector<uint8_t> mask((size_t)std::max<int64_t>(p.n_local, 1), 0);
  for (int q = 0, pi = 0; q < p.world; ++q) {
    if (q == p.rank) continue;
    for (int64_t x = p.send_off[q]; x < p.send_off[q + 1]; ++x)
      mask[(size_t)(all[(size_t)x] - p.row_begin)] |= (uint8_t)(1u << pi);
    ++pi;
  }
  if (p.send_mask) cudaFree(p.send_mask);
  AGNN_CUDA_TRY(cudaMalloc(&p.send_mask, mask.size()));
  AGNN_CUDA_TRY(cudaMemcpy(p.send_mask, mask.data(), mask.size(), cudaMemcpyHostToDevice));
  return AGNN_OK;
}

bool peer_rows(const Plan& p, const void* a, const void* b, PeerRows& out) {
  out = PeerRows();
  if (!p.peer || !p.peer_ready || p.world <= 1) return false;
  PeerPtrs pa, pb;
  if (!peer_lookup(p, a, pa) || (b && !peer_lookup(p, b, pb))) return false;
  for (int q = 0; q < p.world; ++q) {
    if (q == p.rank) continue;
    out.a[out.n] = reinterpret_cast<float*>(pa.p[q]);
    out.b[out.n] = b ? reinterpret_cast<float*>(pb.p[q]) : nullptr;
    ++out.n;
  }
  out.mask = p.send_mask;
  return true;
}

bool peer_out(const Plan& p, const void* c0, const void* c1, PeerOut& out) {
  PeerRows r;
  out = PeerOut();
  if (!peer_rows(p, c0, c1, r)) return false;
  out.n = r.n;
  for (int i = 0; i < r.n; ++i) {
    out.C0[i] = r.a[i];
    out.C1[i] = r.b[i];
  }
  out.mask = r.mask;
  return true;
}

agnn_status nccl_status(ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return AGNN_OK;
  return fail(AGNN_ENCCL, std::string(what) + ": " + ncclGetErrorString(r));
}

agnn_status comm_init(Plan& p, const void* unique_id) {
  if (!unique_id) return peer_init(p);
  ncclUniqueId id;
  memcpy(&id, unique_id, sizeof(id));
  ncclComm_t comm;
  agnn_status st = nccl_status(ncclCommInitRank(&comm, p.world, id, p.rank), "ncclCommInitRank");
  if (st != AGNN_OK) return st;
  p.nccl = comm;
  return AGNN_OK;
}

void comm_destroy(Plan& p) {
  if (p.nccl) ncclCommDestroy(static_cast<ncclComm_t>(p.nccl));
  p.nccl = nullptr;
  if (p.opened) {
    std::lock_guard<std::mutex> lock(g_ipc_mu);
    for (void* q : *p.opened) ipc_release(q);
    delete p.opened;
    p.opened = nullptr;
  }
  delete p.regs;
  p.regs = nullptr;
  if (p.send_idx) cudaFree(p.send_idx);
  p.send_idx = nullptr;
  if (p.send_mask) cudaFree(p.send_mask);
  p.send_mask = nullptr;
  if (p.ctl) cudaFree(p.ctl);
  p.ctl = nullptr;
}

agnn_status allgather_rows(const Plan& p, float* full, int64_t width, cudaStream_t s) {
  const RowArray a{full, width};
  return allgather_rows(p, &a, 1, s);
}

agnn_status allgather_rows(const Plan& p, const RowArray* arrs, int n_arrs, cudaStream_t s) {
  if (p.world <= 1) return AGNN_OK;
  struct Mark {
    cudaStream_t s;
    ~Mark() {
      if (g_profiling) prof_mark("nccl_allgather_rows", s);
    }
  } mark{s};
  if (p.peer) {
    // entry barrier: every peer is done reading its replica (the buffers may be
    // workspace arrays reused by the previous layer); push the rows each peer
    // references; exit barrier
    if (!p.peer_ready) return fail(AGNN_ESTATE, "peer exchange: agnn_plan_connect not called");
    if (n_arrs > 4) return fail(AGNN_EINVAL, "allgather_rows: at most 4 arrays");
    PushArr A;
    A.n = n_arrs;
    for (int i = 0; i < n_arrs; ++i) {
      if (!peer_lookup(p, arrs[i].full, A.dst[i]))
        return fail(AGNN_ESTATE, "peer exchange: buffer not registered (agnn_plan_register)");
      A.src[i] = arrs[i].full;
      A.width[i] = arrs[i].width;
    }
    agnn_status st = peer_barrier(p, s);
    if (st != AGNN_OK) return st;
    const int64_t total = p.send_off[p.world];
    if (total > 0) {
      PeerOffs offs;
      for (int q = 0; q <= p.world; ++q) offs.o[q] = p.send_off[q];
      for (int q = p.world + 1; q <= kMaxPeers; ++q) offs.o[q] = total;
      const int64_t blocks = std::min<int64_t>((total + 7) / 8, (int64_t)kNumSMs * 4);
      peer_push_needed_kernel<<<(unsigned)blocks, 256, 0, s>>>(A, p.send_idx, total, offs);
      AGNN_LAUNCH_CHECK("peer_push_kernel");
    }
    return peer_barrier(p, s);
  }
  ncclComm_t comm = static_cast<ncclComm_t>(p.nccl);
  agnn_status st = nccl_status(ncclGroupStart(), "ncclGroupStart");
  if (st != AGNN_OK) return st;
  for (int i = 0; i < n_arrs; ++i) {
    const int64_t width = arrs[i].width;
    for (int r = 0; r < p.world; ++r) {
      const int64_t rows = p.bounds[r + 1] - p.bounds[r];
      if (rows == 0) continue;
      float* blk = arrs[i].full + p.bounds[r] * width;
      ncclResult_t e = ncclBroadcast(blk, blk, (size_t)(rows * width), ncclFloat32, r, comm, s);
      if (e != ncclSuccess) {
        ncclGroupEnd();
        return nccl_status(e, "ncclBroadcast");
      }
    }
  }
  return nccl_status(ncclGroupEnd(), "ncclGroupEnd");
}

agnn_status allreduce_sum(const Plan& p, float* buf, int64_t count, cudaStream_t s) {
  if (p.world <= 1) return AGNN_OK;
  struct Mark {
    cudaStream_t s;
    ~Mark() {
      if (g_profiling) prof_mark("nccl_allreduce", s);
    }
  } mark{s};
  if (p.peer) {
    if (!p.peer_ready) return fail(AGNN_ESTATE, "peer exchange: agnn_plan_connect not called");
    agnn_status st;
    for (int64_t c0 = 0; c0 < count; c0 += kRedMax) {
      const int64_t cnt = std::min<int64_t>(kRedMax, count - c0);
      const int set = (int)(p.red_calls++ & 1);  // two slot sets: see DESIGN.md §8
      PeerPtrs ctl;
      for (int r = 0; r < p.world; ++r) ctl.p[r] = static_cast<char*>(p.peer_ctl[r]);
      const unsigned blocks = (unsigned)std::min<int64_t>((cnt + 255) / 256, kNumSMs * 4);
      peer_red_write_kernel<<<blocks, 256, 0, s>>>(buf + c0, cnt, ctl, p.rank, p.world, set);
      AGNN_LAUNCH_CHECK("peer_red_write_kernel");
      if ((st = peer_barrier(p, s)) != AGNN_OK) return st;
      peer_red_sum_kernel<<<blocks, 256, 0, s>>>(red_of(p.ctl, p.world, set, 0), cnt, p.world,
                                                  buf + c0);
      AGNN_LAUNCH_CHECK("peer_red_sum_kernel");
    }
    return AGNN_OK;
  }
  return nccl_status(ncclAllReduce(buf, buf, (size_t)count, ncclFloat32, ncclSum,
                                   static_cast<ncclComm_t>(p.nccl), s),
                     "ncclAllReduce");
}

}  // namespace agnn

extern "C" agnn_status agnn_ipc_export(const void* ptr, void* handle, int64_t* offset) {
  using namespace agnn;
  if (!ptr || !handle || !offset) return fail(AGNN_EINVAL, "agnn_ipc_export: NULL argument");
  auto fn = get_range_fn();
  if (!fn) return fail(AGNN_ECUDA, "agnn_ipc_export: cuMemGetAddressRange unavailable");
  CUdeviceptr base = 0;
  size_t size = 0;
  if (fn(&base, &size, (CUdeviceptr)ptr) != CUDA_SUCCESS)
    return fail(AGNN_EINVAL, "agnn_ipc_export: not a device allocation");
  cudaIpcMemHandle_t h;
  AGNN_CUDA_TRY(cudaIpcGetMemHandle(&h, reinterpret_cast<void*>(base)));
  memset(handle, 0, 64);
  memcpy(handle, &h, sizeof(h));
  *offset = (int64_t)((CUdeviceptr)ptr - base);
  return AGNN_OK;
}

extern "C" agnn_status agnn_nccl_unique_id(void* out) {
  if (!out) return agnn::fail(AGNN_EINVAL, "agnn_nccl_unique_id: NULL");
  ncclUniqueId id;
  agnn_status st = agnn::nccl_status(ncclGetUniqueId(&id), "ncclGetUniqueId");
  if (st == AGNN_OK) memcpy(out, &id, sizeof(id));
  return st;
}
