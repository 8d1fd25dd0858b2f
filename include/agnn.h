/*
 * agnn.h — C ABI of the B200-native A-GNN layer hot path (libagnn.so).
 *
 * One layer of an attentional GNN in the paper's global tensor formulation
 * (Besta et al., SC'23, Eq. 1):
 *     H^{l+1} = sigma(Z^l),  Z^l = (Phi o (+))(Psi(A, H^l), H^l)
 * for the three models of PAPER.md:169-177:
 *     AGNN_VA   Psi = A (.) (H H^T)                         (Eq. 7 at :262)
 *     AGNN_AGNN Psi = sm(beta A (.) (H_x (/) n n^T))        (reading A8)
 *     AGNN_GAT  Psi = sm(A (.) LReLU(C)), C = s 1^T + 1 t^T
 * with the graph softmax sm over the stored entries of each row
 * and the backward pass of PAPER.md:221-298
 * (Eq. 2-13; readings A11/A12 in DESIGN.md §2).  The dense n x n virtual
 * matrices are never materialised.
 *
 * Conventions
 *  - Every pointer argument of agnn_forward / agnn_backward / agnn_debug_*
 *    is a DEVICE pointer unless marked "host".  Floating data are fp32,
 *    row-major, 16-byte aligned, rows contiguous (leading dimension = width).
 *  - H_in: [n_local x k_in]; W: [k_in x k_out]; GAT a: [heads][2d] with
 *    a1 = a[h][0:d] (centre vertex = row i), a2 = a[h][d:2d] (neighbour =
 *    column j), d = k_out/heads; H_out, dH_out: [n_local x k_out];
 *    dH_in: [n_local x k_in]; dW: [k_in x k_out]; da: [heads][2d].
 *    AGNN_CGNN: heads == 1, a and da NULL, k_in in 16..256 (multiple of 16).
 *  - The CSR lists, for every local row i, the vertices i aggregates from
 *    (N^(i)), by GLOBAL column id, strictly ascending.
 *    The library computes on exactly this pattern: it never adds self-loops
 *    or symmetrises (use agnn_csr_build for the paper's preprocessing).
 *    With AGNN_CSR_SYMMETRIC ("for undirected graphs A = A^T")
 *    the backward visits every stored entry once for both of its roles.
 *    Without it (a directed pattern, reading A4) the plan builds the
 *    transposed pattern (CSC) once and the backward runs a row pass over the
 *    CSR and a column pass over the CSC; this needs world == 1 and the plan
 *    holding every row (agnn_backward returns AGNN_EUNSUPPORTED otherwise).
 *
 * Ownership
 *  - The caller owns every feature, weight, gradient, `saved` and
 *    `workspace` buffer (sizes from agnn_saved_bytes / agnn_workspace_bytes).
 *    The plan owns only derived metadata (work lists, NCCL communicator);
 *    the model owns nothing on the device.
 *  - agnn_forward / agnn_backward never allocate, never synchronise the
 *    host and only enqueue work on `stream`: they are CUDA-graph capturable
 *    when world == 1.
 *
 * Errors
 *  - Every call returns an agnn_status; C++ exceptions never cross the ABI.
 *    agnn_last_error() returns a thread-local message for the last failure.
 *  - Descriptor / argument checks on the host return AGNN_EINVAL (e.g.
 *    k_out % heads != 0, unsupported widths, misaligned pointers).
 *  - CSR content errors (non-monotone row_ptr, column out of range,
 *    unsorted or duplicate columns) are detected on the device and surface
 *    ONLY from agnn_plan_create (the one call that synchronises).
 *  - CUDA launch failures return AGNN_ECUDA, NCCL failures AGNN_ENCCL.
 *  - With world > 1 every rank must call forward/backward in the same order.
 */
#ifndef AGNN_H
#define AGNN_H

#include <stddef.h>
#include <stdint.h>
#include <cuda_runtime.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  AGNN_OK = 0,
  AGNN_EINVAL = 1,
  AGNN_ECUDA = 2,
  AGNN_ENCCL = 3,
  AGNN_ENOMEM = 4,
  AGNN_EUNSUPPORTED = 5,
  AGNN_ESTATE = 6
} agnn_status;

/* AGNN_CGNN: a C-GNN layer sigma((A (x) H) W), the aggregation a
 * matrix product over the semiring `agg` (S§8(f) f3)        */
typedef enum { AGNN_VA = 0, AGNN_AGNN = 1, AGNN_GAT = 2, AGNN_CGNN = 3 } agnn_kind;

/* C-GNN aggregation (readings C1-C4), d_i = stored entries of row i:
 *   SUM  X_i = sum_{j in N(i)} H_j               (real semiring)
 *   MEAN X_i = sum_j H_j / d_i                   (averaging semiring)
 *   GCN  X_i = sum_j H_j / sqrt(d_i d_j)         (normalised A)
 *   MAX / MIN  X_ic = max / min_j H_jc           (tropical semirings);
 *        an empty row gives 0; the gradient goes to the smallest j among ties */
typedef enum {
  AGNN_AGG_SUM = 0,
  AGNN_AGG_MEAN = 1,
  AGNN_AGG_GCN = 2,
  AGNN_AGG_MAX = 3,
  AGNN_AGG_MIN = 4
} agnn_agg;

/* sigma; reading A6: ReLU with sigma'(0) = 0, ELU(alpha = 1) */
typedef enum { AGNN_ACT_NONE = 0, AGNN_ACT_RELU = 1, AGNN_ACT_ELU = 2 } agnn_act;

/* precision mode.  Arithmetic is fp32 everywhere (dense projection: fp32 FFMA
 * or 3xTF32 on tcgen05, both fp32-accurate; sparse passes: fp32 FMA).
 * AGNN_PREC_BF16 (GAT, k_out = 128, heads 1/2/4/8, symmetric pattern):
 * the gathered feature rows are STORED as bfloat16 — the projection P = HW
 * (rounded to nearest-even from the fp32 GEMM result; the scores s, t come from
 * the unrounded product, a' = Wa being its own GEMM column) and
 * the backward's G = dH_out (.) sigma'(Z) (rounded, then used throughout:
 * delta, dalpha, the aggregation of G).  Everything else (H, Z, H_out, dP, dW,
 * da, dH, the saved statistics) stays fp32.  This is north_star's "BF16
 * projection" mode, tolerance 1e-2 normwise (reading B1); it halves
 * the bytes of every gather.
 * AGNN / VA (k_in = 128 / 256, symmetric pattern; reading B2): the gathered
 * operands are the layer input and the backward's M = G W^T, so the layer
 * computes on H~ = bf16(H) throughout (scores, norms nu, aggregation X = Psi H~)
 * and the backward uses M~ = bf16(M) (rounded in the GEMM epilogue); X, Z, G,
 * dW, dH and all statistics are fp32.  Other shapes: AGNN_EUNSUPPORTED.      */
typedef enum {
  AGNN_PREC_FP32 = 0,    /* fp32 FFMA, or 3xTF32 on tcgen05 (fp32-accurate)  */
  AGNN_PREC_TF32X3 = 1,  /* same arithmetic as FP32 (the tcgen05 path is used wherever it has a shape) */
  AGNN_PREC_BF16 = 2     /* GAT: P, G stored as bf16 (B1); AGNN/VA: H, M (B2) */
} agnn_prec;

/* agnn_csr.flags.
 * AGNN_CSR_SYMMETRIC: the pattern is symmetric ("for undirected
 *   graphs A = A^T"); the backward then visits every stored entry once for
 *   both of its roles.  The library trusts the flag unless
 * AGNN_PLAN_VERIFY_SYMMETRY is also set: agnn_plan_create then checks on the
 *   device that every stored (i,j) has its transpose (j,i) stored, and returns
 *   AGNN_EINVAL if one is missing (world == 1 with every row in the plan; with
 *   world > 1 each rank can see only its own rows, so the flag makes
 *   agnn_plan_create return AGNN_EUNSUPPORTED).  Costs one binary search per
 *   stored entry at plan time; nothing at run time.                         */
enum { AGNN_CSR_SYMMETRIC = 1u, AGNN_PLAN_VERIFY_SYMMETRY = 2u };

typedef struct {
  int64_t n;               /* global vertex count                                  */
  int64_t row_begin;       /* this rank owns global rows [row_begin, row_end)      */
  int64_t row_end;
  const int64_t* row_ptr;  /* device, [row_end - row_begin + 1], row_ptr[0] == 0   */
  const int32_t* col_idx;  /* device, [row_ptr[n_local]], global ids, ascending    */
  uint32_t flags;          /* AGNN_CSR_SYMMETRIC | AGNN_PLAN_VERIFY_SYMMETRY       */
} agnn_csr;

/* Work-decomposition options of a plan (agnn_plan_create_ex).  None of them
 * changes what is computed: every choice gives the same outputs up to fp32
 * rounding order (the chunk size fixes the summation order of heavy rows, so a
 * plan with a different chunk size is a different, equally valid rounding).
 * A field < 0 (or 0 for chunk_edges) takes the default; agnn_plan_create uses
 * all defaults.  Values out of range return AGNN_EINVAL.                     */
typedef struct {
  int32_t chunk_edges;    /* heavy-row chunk size in stored entries, 32 .. 2^30;
                             default: 256 for n <= 2^21, doubling per doubling of
                             n, at most 2048 (a function of the global n only)  */
  int32_t short_edges;    /* rows of degree <= short_edges go to the short-row
                             kernels where a kernel has one; 0 .. 32, default 32  */
  int32_t short_bundles;  /* GAT k'=128 short rows packed into 32-entry warp
                             bundles: 0 never, 1 fp32 storage only (default),
                             2 fp32 and bf16                                       */
  int32_t gat_factored;   /* GAT factored backward: 0 never,
                             1 k_out = 128 only (default), 2 every width          */
  int32_t l2_hot_mb;      /* L2 budget (MB) of the evict_last gathers, 0 disables
                             the hints; default 96 (performance only, see below)  */
  int32_t spmmm;          /* AGNN/VA forward with k_in = k_out = 128: 1 fuses the
                             aggregation and the projection into one SpMMM kernel
                             (Table 2; X = Psi H goes to the
                             tensor core through shared memory, not HBM), 0 runs
                             the SpMM kernel and then the tcgen05 GEMM; default 0
                             (measured).  Outputs agree up to fp32
                             rounding order.                                      */
} agnn_plan_options;

typedef struct {
  int rank, world;
  const void* nccl_unique_id; /* host, 128 bytes (ncclUniqueId): NCCL exchange; NULL:
                                 peer-memory exchange (world <= 8, see agnn_plan_connect) */
  const int64_t* bounds;      /* host, [world + 1] row bounds (agnn_partition)      */
} agnn_dist;

typedef struct {
  agnn_kind kind;
  int k_in, k_out, heads;  /* GAT: heads >= 1, k_out % heads == 0; AGNN/VA: heads == 1 */
  agnn_act act;
  agnn_prec prec;
  float negative_slope;    /* GAT LeakyReLU slope lambda (reading A5), 0.2          */
  float beta;              /* AGNN temperature (reading A8), 1.0, not trained        */
  float eps;               /* AGNN norm floor nu_i = max(||h_i||, eps), 1e-12        */
  agnn_agg agg;            /* C-GNN aggregation semiring (ignored by the A-GNNs)     */
} agnn_layer_desc;

typedef struct agnn_plan_s* agnn_plan_t;
typedef struct agnn_model_s* agnn_model_t;

/* 1D row-block partition (reading A20; the paper's own scheme is 2D,
 * PAPER.md:321).  Pure host function, bit-exact with the oracle:
 * w(r) = row_ptr[r] + c_v * r, bounds[0] = 0, bounds[world] = n,
 * bounds[p] = min{ r : w(r) >= ceil(p * w(n) / world) }.  row_ptr is host. */
agnn_status agnn_partition(int64_t n, const int64_t* row_ptr_host, int world, int64_t c_v,
                           int64_t* bounds_host);

/* Validate the CSR on the device, build the work lists (light rows + heavy-row
 * chunks, short-row bundles), and (world > 1) create the NCCL communicator.
 * Also builds the L2 residency classes of the columns: a plan-owned copy of
 * col_idx (nnz x 4 bytes of device memory) whose free high bits rank every
 * column by how often this rank gathers it; the sparse kernels load the rows of
 * the most-gathered columns with an evict_last L2 policy (
 * agnn_plan_options.l2_hot_mb).  The classes are performance metadata only:
 * no result depends on them.  With world == 1 the CSR must hold every row
 * (row_begin == 0, row_end == n), else AGNN_EINVAL.  Synchronises. */
agnn_status agnn_plan_create(const agnn_csr* csr, const agnn_dist* dist /* NULL => 1 GPU */,
                             cudaStream_t stream, agnn_plan_t* out);
/* The same with explicit work-decomposition options (NULL => defaults).      */
agnn_status agnn_plan_create_ex(const agnn_csr* csr, const agnn_dist* dist,
                                const agnn_plan_options* options, cudaStream_t stream,
                                agnn_plan_t* out);
agnn_status agnn_plan_destroy(agnn_plan_t plan);
/* host-side statistics (info: 12 int64, host): [0]=n_local [1]=nnz_local
 * [2]=light rows [3]=heavy rows [4]=heavy chunks [5]=chunk size [6]=max degree
 * [7]=n (global) [8]=short rows (light rows of degree <= [9], taken by the
 * short-row kernels where a kernel has one) [9]=short_max
 * (agnn_plan_options.short_edges; 0: no split) [10]=rows of other blocks this
 * rank's rows reference (received per peer-memory exchange) [11]=rows of this
 * rank's block sent per peer-memory exchange (summed over the peers; known after
 * agnn_plan_connect) */
agnn_status agnn_plan_info(agnn_plan_t plan, int64_t* info);

/* The transposed pattern of the plan's CSR (test/utility; synchronises):
 * col_ptr [n+1] (device, int64), row_idx [nnz] (device, int32) list, for
 * every column j, the rows i with a stored entry (i,j) in ascending i, and
 * perm [nnz] (device, int64, nullable) the CSR position of each CSC entry.
 * Requires world == 1 and the plan holding all rows (else AGNN_EUNSUPPORTED). */
agnn_status agnn_plan_csc(agnn_plan_t plan, int64_t* col_ptr, int32_t* row_idx, int64_t* perm,
                          cudaStream_t stream);

agnn_status agnn_model_create(agnn_plan_t plan, int n_layers, const agnn_layer_desc* descs,
                              agnn_model_t* out);
agnn_status agnn_model_destroy(agnn_model_t model);

/* bytes of the per-layer `saved` buffer (intermediates kept for backward)
 * and of the scratch `workspace` shared by forward and backward.  For GAT with
 * k_out = 128 on a symmetric pattern `saved` also holds Q [n_local x k_out]
 * (the factored backward: ds_j = G_j . Q_j); the layout is
 * internal, only the size is part of the contract.                          */
agnn_status agnn_saved_bytes(agnn_model_t model, int layer, size_t* bytes);
agnn_status agnn_workspace_bytes(agnn_model_t model, int layer, size_t* bytes);

/* Layer forward: H_out = sigma(Z).  saved == NULL => inference mode (nothing
 * kept, PAPER.md:623/:636 --inference); otherwise `saved` receives what
 * agnn_backward needs.  Enqueued on `stream`.                              */
agnn_status agnn_forward(agnn_model_t model, int layer, const float* W, const float* a,
                         const float* H_in, float* H_out, void* saved, void* workspace,
                         cudaStream_t stream);

/* Layer backward (Eq. 6): from dH_out = dL/dH^{l+1} computes
 * dH_in = Gamma = dL/dH^l (nullable: skipped), dW = Y^l, and for GAT
 * da = dL/da (reading A12; NULL for VA/AGNN).  `saved` is the buffer filled
 * by the matching agnn_forward; H_in is the same layer input.              */
agnn_status agnn_backward(agnn_model_t model, int layer, const float* W, const float* a,
                          const float* H_in, const void* saved, const float* dH_out,
                          float* dH_in, float* dW, float* da, void* workspace,
                          cudaStream_t stream);

/* ---- the steps either side of the layer path in a training loop --------- */
/* Loss of reading A13, L = <R, H> = sum_e R[e] * H[e] over `count` fp32
 * elements (R = dL/dH^L, the Eq. 4 bootstrap).  scratch: device,
 * AGNN_LOSS_SCRATCH doubles; *loss: device double (this rank's rows only: with
 * world > 1 the caller adds the ranks' values).  Deterministic fixed-order
 * fp64 reduction.  R, H 16-byte aligned.                                     */
#define AGNN_LOSS_SCRATCH 1024
agnn_status agnn_loss_inner(const float* R, const float* H, int64_t count, double* scratch,
                            double* loss, cudaStream_t stream);
/* SGD update of PAPER.md:244: W[e] -= lr * dW[e] for e < count (device).    */
agnn_status agnn_sgd_step(float* W, const float* dW, int64_t count, float lr,
                          cudaStream_t stream);

/* Test-only export (excluded from timing): recompute the attention
 * coefficients alpha of `count` stored entries (positions into the LOCAL
 * col_idx) from the saved row statistics.  alpha_out: [count x heads].
 * GAT/AGNN give the softmax alpha_ij, VA the raw score S_ij.  H_in is the
 * layer input (needed by AGNN/VA on one GPU; ignored for GAT).             */
agnn_status agnn_debug_attention(agnn_model_t model, int layer, const void* saved,
                                 const float* H_in, const int64_t* edge_pos, int64_t count,
                                 float* alpha_out, cudaStream_t stream);

/* Test-only export: C[M x N] = A[M x K] B^T with B given as [N x K], through the
 * same dense-projection path the layers use (tcgen05 3xTF32 when the shape has
 * an instantiation, else fp32 FFMA).  Device pointers, row-major.          */
agnn_status agnn_debug_gemm(const float* A, int64_t M, int K, const float* B, int N, float* C,
                            cudaStream_t stream);

/* Test-only export: C[K1 x N] = A^T B over the M rows of A [M x K1] and
 * B [M x N] (the weight-gradient contraction, Eq. 5), with the
 * split partials in `ws` (agnn_debug_gemm_tn_ws_bytes bytes, device).       */
agnn_status agnn_debug_gemm_tn(const float* A, int64_t M, int K1, const float* B, int N, float* C,
                               float* ws, cudaStream_t stream);
size_t agnn_debug_gemm_tn_ws_bytes(int K1, int N);

/* Number of kernels this library launched since load (all entry points).   */
uint64_t agnn_launch_count(void);

/* Live per-kernel timing for the bench (off by default).  When enabled, a CUDA
 * event is recorded on the launch stream after every kernel (and at the start
 * of each forward/backward call); a kernel's time is the gap to the previous
 * event on that stream.  report() synchronises on the recorded events and
 * writes "name launches total_ms" lines into buf (host, len bytes).        */
agnn_status agnn_profile_enable(int on);
agnn_status agnn_profile_report(char* buf, size_t len);
agnn_status agnn_profile_reset(void);
/* ---- peer-memory exchange (world > 1, agnn_dist.nccl_unique_id == NULL) ----
 * The ranks' replicated buffers are mapped into each other with CUDA IPC
 * (loads / stores over NVLink / NVSwitch; S§8(e)).  Setup, once per plan (host,
 * synchronising; the caller moves the 64-byte handles between ranks, e.g. with
 * torch.distributed all_gather_object):
 *   1. agnn_plan_ctl_export on every rank, all-gather, agnn_plan_connect;
 *   2. for every `saved` and `workspace` buffer passed to forward/backward:
 *      agnn_ipc_export on every rank, all-gather, agnn_plan_register.
 * Every rank must register its buffers in the same order with the same sizes.
 * handles: [world][64 B] in rank order; offsets: [world] byte offsets of the
 * buffer inside each rank's allocation (both host).                          */
agnn_status agnn_ipc_export(const void* device_ptr, void* handle64, int64_t* offset);
agnn_status agnn_plan_ctl_export(agnn_plan_t plan, void* handle64, int64_t* offset);
agnn_status agnn_plan_connect(agnn_plan_t plan, const void* handles, const int64_t* offsets);
agnn_status agnn_plan_register(agnn_plan_t plan, void* local, size_t bytes, const void* handles,
                               const int64_t* offsets);

/* ncclGetUniqueId for the multi-GPU plan (host, 128 bytes).                 */
agnn_status agnn_nccl_unique_id(void* out128);

/* ---- utilities (harness / tests; not on the timed path) ---------------- */
enum { AGNN_BUILD_SYMMETRIZE = 1u, AGNN_BUILD_SELF_LOOPS = 2u, AGNN_BUILD_CONNECT_ISOLATED = 4u };

/* Canonical CSR (readings A1-A3, A21) from n_pairs device edge samples:
 * drop self-pairs, optionally symmetrise, dedup, optionally connect every
 * vertex without a non-self neighbour to (v+1) mod n (both directions),
 * optionally add (v,v) for all v.  row_ptr: device [n+1], caller-allocated;
 * *col_idx: device, allocated by the library (free with agnn_free);
 * *nnz_out: host.  Uses device radix sort; synchronises.                   */
agnn_status agnn_csr_build(int64_t n, const uint32_t* src, const uint32_t* dst, int64_t n_pairs,
                           uint32_t build_flags, int64_t* row_ptr, int32_t** col_idx,
                           int64_t* nnz_out, cudaStream_t stream);
void agnn_free(void* device_ptr);

const char* agnn_status_string(agnn_status status);
const char* agnn_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* AGNN_H */
