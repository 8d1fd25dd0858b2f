// internal.cuh — launcher prototypes shared between the .cu files of libagnn.so
#pragma once
#include "common.cuh"

namespace agnn {

// ---- work items (plan) ---------------------------------------------------------
struct Items {
  const int64_t* row_ptr;     // local rows
  const int32_t* col;         // global column ids
  const int32_t* light_rows;  // local row ids
  int64_t n_light;
  const int32_t* chunk_row;
  const int32_t* chunk_idx;
  int64_t n_chunks;
  int chunk;
  const int32_t* heavy_rows;
  const int32_t* heavy_off;
  int64_t n_heavy;
  int64_t row_begin;          // global id of local row 0
  int64_t n_local;
  // the light rows split by degree (kernels with a short-row variant): rows of degree
  // <= the plan's short_max (short) and the others (long); items_of_csc: none
  const int32_t* short_rows;
  const int4* short_meta;     // per short row {row, degree, beg lo, beg hi}; non-empty first
  int64_t n_short;
  int64_t n_short_nz;         // short rows with stored entries
  const int4* bundles;        // {first short record, rows, entries, 0} (gat_short.cu)
  int64_t n_bundles;
  const int32_t* long_rows;
  int64_t n_long;
  // L2 residency hints (see l2_hinted): col entries carry the column class in the
  // bits above col_mask; a gathered row is loaded with evict_last iff its entry
  // (class bits included) is >= hot_thr, else with evict_first (cold_first) or normal
  uint32_t col_mask = 0x7fffffffu;
  uint32_t hot_thr = 0xffffffffu;
  int cold_first = 0;
  int bundle_mode = 1;        // the plan's short-row bundle mode (gat_bundles_enabled)
};
constexpr int kMaxColClasses = 64;
// the items `it` of plan `p` with L2 hints for gathered rows of `row_bytes` bytes
// per pass (the hot class is the largest set of rows that fits the L2 budget)
Items l2_hinted(const Items& it, const Plan& p, int64_t row_bytes);
// device side of the hints: decode a (possibly classed) column entry c >= 0 into the
// row id and the L2 policy of its gather
struct Gath {
  uint32_t mask, thr;
  L2Pol pol;
  __device__ __forceinline__ explicit Gath(const Items& it)
      : mask(it.col_mask), thr(it.hot_thr), pol(make_l2pol(it.cold_first)) {}
  __device__ __forceinline__ Gath(uint32_t m, uint32_t t, int cf)
      : mask(m), thr(t), pol(make_l2pol(cf)) {}
  __device__ __forceinline__ int64_t row(int c) const { return (int64_t)((uint32_t)c & mask); }
  __device__ __forceinline__ uint64_t policy(int c) const {
    return (uint32_t)c >= thr ? pol.hot : pol.cold;
  }
};
Items items_of(const Plan& p);
// the transposed pattern's items (directed plans): "rows" are columns j, col = rows i
Items items_of_csc(const Plan& p);
// CSC (+ optional CSR position of every CSC entry) of a local CSR with n_rows rows
// starting at global row 0; device radix sort, synchronises (plan time only)
agnn_status build_csc(const int64_t* row_ptr, const int32_t* col, int64_t n_rows, int64_t n,
                      int64_t nnz, int64_t* csc_ptr, int32_t* csc_idx, int64_t* perm,
                      cudaStream_t s);


// persistent sparse-kernel grid: 256-thread blocks, SMs x resident blocks of `func`
constexpr int kSparseThreads = 256;
constexpr int kMaxSparseBlocks = kNumSMs * 8;
int persistent_blocks(const void* func);
template <typename F>
inline int grid_of(F* func) { return persistent_blocks(reinterpret_cast<const void*>(func)); }

// ---- GEMMs (gemm_simt.cu) -----------------------------------------------------
// C[M x N] = A[M x K] * op(B);  op(B) = B ([K x N], ldb=N) or B^T (B is [N x K]).
// Columns [0, n_split) go to C0 (ld = n_split), [n_split, N) to C1 (ld = N - n_split).
// If Cact != NULL, sigma(C) (act) is also written to Cact (layout of C0); C0 may be NULL.
// Columns >= n_store (padding) are computed but not stored (n_store <= 0: N).
// replicas of up to two row arrays in the other ranks (compact peer order: rank order
// without this rank) and the needed-rows mask: local row r goes to peer pi iff bit pi
// of mask[r] is set (the fused exchange; kernel argument, unused when n = 0)
struct PeerRows {
  int n = 0;
  float* a[kMaxPeers - 1] = {};
  float* b[kMaxPeers - 1] = {};
  const uint8_t* mask = nullptr;
};
// the same for a GEMM's output column blocks C0 | C1 (gemm_rows)
struct PeerOut {
  int n = 0;
  float* C0[kMaxPeers - 1] = {};
  float* C1[kMaxPeers - 1] = {};
  const uint8_t* mask = nullptr;
};
agnn_status gemm_rows(const float* A, int64_t M, int K, const float* B, bool b_trans, int N,
                      float* C0, int n_split, float* C1, cudaStream_t s, float* Cact = nullptr,
                      int act = 0, int n_store = 0, const PeerOut* peers = nullptr,
                      bool* peers_done = nullptr);
// peer exchange: the fused-exchange descriptors of replicated arrays (compact peer
// order + the plan's needed-rows mask); false if the plan has no peer exchange
bool peer_rows(const Plan& p, const void* a, const void* b, PeerRows& out);
bool peer_out(const Plan& p, const void* c0, const void* c1, PeerOut& out);
// BF16 storage (reading B1): C = A * B^T with columns [0, n_split) rounded to bf16
// into C0h (ld n_split) and [n_split, N) fp32 into C1 (ld N - n_split); scratch
// [M x n_split] fp32 is used only when the shape has no tcgen05 instantiation.
agnn_status gemm_rows_bf16(const float* A, int64_t M, int K, const float* B, int N, bf16* C0h,
                           int n_split, float* C1, float* scratch, cudaStream_t s);
// C[K1 x N] = A^T B over M rows (A [M x K1], B [M x N]); deterministic split-M with
// partials in `ws` (gemm_tn_ws_floats) and an ordered reduction.  If accumulate,
// C += result.
size_t gemm_tn_ws_floats(int K1, int N);
// Y[cols x rows] = X[rows x cols]^T (small weight matrices)
agnn_status transpose(const float* X, int rows, int cols, float* Y, cudaStream_t s);
agnn_status gemm_tn(const float* A, int64_t M, int K1, const float* B, int N, float* C,
                    float* ws, cudaStream_t s);

// ---- GAT (gat.cu) ---------------------------------------------------------------
struct GatShape {
  int k_in, k_out, heads;
  float slope;
  int act;
  bool bf16;  // AGNN_PREC_BF16: P and G stored as bfloat16 (reading B1)
};
size_t gat_saved_bytes(const Plan& p, const GatShape& g);
size_t gat_workspace_bytes(const Plan& p, const GatShape& g);
agnn_status gat_forward(const Plan& p, const GatShape& g, const float* W, const float* a,
                        const float* H_in, float* H_out, void* saved, void* ws, cudaStream_t s);
agnn_status gat_backward(const Plan& p, const GatShape& g, const float* W, const float* a,
                         const float* H_in, const void* saved, const float* dH_out,
                         float* dH_in, float* dW, float* da, void* ws, cudaStream_t s);
agnn_status gat_debug_alpha(const Plan& p, const GatShape& g, const void* saved,
                            const int64_t* edge_pos, int64_t count, float* out, cudaStream_t s);

// ---- multi-GPU exchange (comm.cu) -------------------------------------------------
// all-gather of row blocks: rows [bounds[r], bounds[r+1]) of `full` (row width
// `width` floats) are broadcast from rank r; in place.
// Peer transport: only the rows each peer's CSR references are sent (comm.cu).
agnn_status allgather_rows(const Plan& p, float* full, int64_t width, cudaStream_t s);
struct RowArray {
  float* full;     // replicated [n x width] array (rows of this rank's block are sent)
  int64_t width;   // floats per row
};
// several arrays in one exchange (one barrier pair, one push kernel); n_arrs <= 4
agnn_status allgather_rows(const Plan& p, const RowArray* arrs, int n_arrs, cudaStream_t s);
// agnn_plan_connect: the send lists from the peers' wanted columns
agnn_status peer_send_lists(Plan& p);
agnn_status allreduce_sum(const Plan& p, float* buf, int64_t count, cudaStream_t s);
agnn_status comm_init(Plan& p, const void* unique_id);  // unique_id NULL: peer-memory exchange
// peer-memory exchange helpers (comm.cu)
agnn_status peer_barrier(const Plan& p, cudaStream_t s);
// map every rank's IPC handle (rank order, 64 B each) + byte offset; own rank -> local
agnn_status peer_open(Plan& p, const void* handles, const int64_t* offsets, void* local,
                      char* out[kMaxPeers]);
// the addresses of `local` (inside a registered buffer) in every rank's copy
agnn_status peer_targets(const Plan& p, const void* local, void* out[kMaxPeers]);
void comm_destroy(Plan& p);

}  // namespace agnn
