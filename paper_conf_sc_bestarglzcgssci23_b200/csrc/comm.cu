// comm.cu — the multi-GPU exchange steps of the 1D row-block layout.
//
// The paper distributes A-stationary 1.5D/2D blocks over MPI; on
// one NVSwitch box every GPU reaches every peer at full bandwidth, so the build
// uses contiguous row blocks: rank r owns rows [bounds[r], bounds[r+1]) and the
// only exchanges are
//   forward : all-gather of the projected rows (P | s t) or (H | nu)
//   backward: all-gather of G (or M) plus per-vertex records
//             all-reduce of the weight gradients dW, da
// The variable-size all-gather is a group of ncclBroadcast calls (one root per
// rank, in place), since NCCL has no all-gather-v.
#include <nccl.h>

#include "internal.cuh"

namespace agnn {

agnn_status nccl_status(ncclResult_t r, const char* what) {
  if (r == ncclSuccess) return AGNN_OK;
  return fail(AGNN_ENCCL, std::string(what) + ": " + ncclGetErrorString(r));
}

agnn_status comm_init(Plan& p, const void* unique_id) {
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
}

agnn_status allgather_rows(const Plan& p, float* full, int64_t width, cudaStream_t s) {
  if (p.world <= 1) return AGNN_OK;
  struct Mark {
    cudaStream_t s;
    ~Mark() {
      if (g_profiling) prof_mark("nccl_allgather_rows", s);
    }
  } mark{s};
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
  return nccl_status(ncclAllReduce(buf, buf, (size_t)count, ncclFloat32, ncclSum,
                                   static_cast<ncclComm_t>(p.nccl), s),
                     "ncclAllReduce");
}

}  // namespace agnn

extern "C" agnn_status agnn_nccl_unique_id(void* out) {
  if (!out) return agnn::fail(AGNN_EINVAL, "agnn_nccl_unique_id: NULL");
  ncclUniqueId id;
  agnn_status st = agnn::nccl_status(ncclGetUniqueId(&id), "ncclGetUniqueId");
  if (st == AGNN_OK) memcpy(out, &id, sizeof(id));
  return st;
}
