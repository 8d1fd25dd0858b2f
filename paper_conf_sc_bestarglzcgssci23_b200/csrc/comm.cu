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
//    agnn_plan_register); an all-gather is a kernel that stores this rank's rows
//    straight into every peer's replica, fenced by a flag barrier; an all-reduce
//    writes this rank's partial into every peer's slot and each rank adds the
//    slots in rank order (identical, deterministic result on every rank).  The
//    projection GEMM can also store its output rows into the peers' replicas
//    from its epilogue (gat.cu), so that exchange overlaps the GEMM tile by tile.
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

// rows [off, off + count) of a replicated array: local copy -> every peer's copy
__global__ void peer_push_kernel(const float* __restrict__ src, PeerPtrs dst, int rank, int world,
                                 int64_t off, int64_t count) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const bool vec = ((off | count) & 3) == 0;
  if (vec) {
    for (int64_t i = t0; i < count / 4; i += stride) {
      const float4 v = ldg4(src + off + 4 * i);
      for (int r = 0; r < world; ++r)
        if (r != rank) st4(reinterpret_cast<float*>(dst.p[r]) + off + 4 * i, v);
    }
  } else {
    for (int64_t i = t0; i < count; i += stride) {
      const float v = src[off + i];
      for (int r = 0; r < world; ++r)
        if (r != rank) reinterpret_cast<float*>(dst.p[r])[off + i] = v;
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

agnn_status peer_init(Plan& p) {
  p.peer = true;
  p.regs = new std::vector<Plan::Reg>();
  p.opened = new std::vector<void*>();
  AGNN_CUDA_TRY(cudaMalloc(&p.ctl, ctl_bytes(p.world)));
  AGNN_CUDA_TRY(cudaMemset(p.ctl, 0, ctl_bytes(p.world)));
  AGNN_CUDA_TRY(cudaDeviceSynchronize());
  return AGNN_OK;
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
  if (p.ctl) cudaFree(p.ctl);
  p.ctl = nullptr;
}

agnn_status allgather_rows(const Plan& p, float* full, int64_t width, cudaStream_t s) {
  if (p.world <= 1) return AGNN_OK;
  struct Mark {
    cudaStream_t s;
    ~Mark() {
      if (g_profiling) prof_mark("nccl_allgather_rows", s);
    }
  } mark{s};
  if (p.peer) {
    // entry barrier: every peer is done reading its replica of `full` (the buffer
    // may be a workspace array reused by the previous layer); push; exit barrier
    if (!p.peer_ready) return fail(AGNN_ESTATE, "peer exchange: agnn_plan_connect not called");
    PeerPtrs dst;
    if (!peer_lookup(p, full, dst))
      return fail(AGNN_ESTATE, "peer exchange: buffer not registered (agnn_plan_register)");
    agnn_status st = peer_barrier(p, s);
    if (st != AGNN_OK) return st;
    const int64_t off = p.row_begin * width, count = p.n_local * width;
    if (count > 0) {
      const int64_t blocks = std::min<int64_t>((count / 4 + 255) / 256 + 1, (int64_t)kNumSMs * 8);
      peer_push_kernel<<<(unsigned)blocks, 256, 0, s>>>(full, dst, p.rank, p.world, off, count);
      AGNN_LAUNCH_CHECK("peer_push_kernel");
    }
    return peer_barrier(p, s);
  }
  ncclComm_t comm = static_cast<ncclComm_t>(p.nccl);
  agnn_status st = nccl_status(ncclGroupStart(), "ncclGroupStart");
  if (st != AGNN_OK) return st;
  for (int r = 0; r < p.world; ++r) {
    const int64_t rows = p.bounds[r + 1] - p.bounds[r];
    if (rows == 0) continue;
    float* blk = full + p.bounds[r] * width;
    ncclResult_t e = ncclBroadcast(blk, blk, (size_t)(rows * width), ncclFloat32, r, comm, s);
    if (e != ncclSuccess) {
      ncclGroupEnd();
      return nccl_status(e, "ncclBroadcast");
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
