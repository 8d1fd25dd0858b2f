/*
 * agnn_oracle.c — FP64 CPU ORACLE for the A-GNN layer hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.
 * The product path (libagnn.so + the Python binding) never links, imports or
 * calls anything here, and this file shares no code, header, table or helper
 * with paper_conf_sc_bestarglzcgssci23_b200/csrc/.
 *
 * What it computes: the plain edge-by-edge LOCAL formulation of one A-GNN
 * layer, forward and backward, in double precision, following
 *   PAPER.md:77-79  (§1, GAT local formula: softmax over N^(v) of
 *                    sigma(a^T [W h_v || W h_u]))
 *   PAPER.md:121    (§2.2, h_i^{l+1} = phi(h_i, (+)_{j in N(i)} psi(h_i, h_j)))
 *   PAPER.md:164    (§4 Eq. 1, H^{l+1} = sigma(Z^l), Z = (Phi o (+))(Psi(A,H),H))
 *   PAPER.md:173-177 (§4.1, Psi for VA, AGNN, GAT)
 *   PAPER.md:191    (§4.2, softmax over the non-zeros of each row)
 *   PAPER.md:221-254 (§5.1-5.2 Eq. 2-6, G = dL/dZ, Y = dL/dW)
 *   PAPER.md:262-298 (§5.3 Eq. 7-13, VA backward)
 * and the readings A1-A22 listed in DESIGN.md §2.
 * Every loop below is a direct transcription of those per-edge definitions;
 * no blocking, fusion or reordering.  OpenMP only splits independent rows
 * (or, for column sums, independent columns via an explicitly built CSC).
 *
 * Conventions: H is n x k row-major, W is k x kout row-major (Z = H W or
 * Z = X W), GAT a is [heads][2d] with a1 = a[h][0:d] (centre v = row i) and
 * a2 = a[h][d:2d] (neighbour u = column j), d = kout / heads.
 * act: 0 = identity, 1 = ReLU (sigma'(0) = 0), 2 = ELU(alpha = 1).
 *
 * Parity pins: every function here is pinned by tests/test_oracle_pins.py
 * (dense global formulation via autograd, finite differences, the paper's VA
 * closed forms Eq. 7/11/12/13, complete-graph / uniform-attention special
 * cases, permutation equivariance, multi-head = concatenation, CSR brute
 * force, partition brute force).  No function is "parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ */
/* activation sigma and its derivative (PAPER.md:164 Eq. 1, :224 Step 2) */
static double act_f(int act, double z) {
  if (act == 1) return z > 0.0 ? z : 0.0;
  if (act == 2) return z > 0.0 ? z : exp(z) - 1.0;
  return z;
}
static double act_df(int act, double z) {
  if (act == 1) return z > 0.0 ? 1.0 : 0.0;
  if (act == 2) return z > 0.0 ? 1.0 : exp(z);
  return 1.0;
}

/* ------------------------------------------------------------------ */
/* Canonical CSR (readings A1-A3, A21).  Pairs (src,dst): self-pairs are
 * dropped; flag 1 adds the reverse of every pair; duplicates are removed;
 * flag 4 then connects every vertex v with no non-self neighbour to
 * (v+1) mod n in both directions; flag 2 adds (v,v) for every v.
 * Rows ascending, columns strictly ascending within a row.              */
static int cmp_u64(const void* x, const void* y) {
  uint64_t a = *(const uint64_t*)x, b = *(const uint64_t*)y;
  return a < b ? -1 : a > b ? 1 : 0;
}
static int64_t sort_unique(uint64_t* keys, int64_t cnt) {
  qsort(keys, (size_t)cnt, sizeof(uint64_t), cmp_u64);
  int64_t w = 0;
  for (int64_t i = 0; i < cnt; ++i)
    if (w == 0 || keys[i] != keys[w - 1]) keys[w++] = keys[i];
  return w;
}

int64_t oracle_csr_capacity(int64_t n, int64_t n_pairs) { return 2 * n_pairs + 3 * n; }

int oracle_csr_build(int64_t n, const uint32_t* src, const uint32_t* dst, int64_t n_pairs,
                     uint32_t flags, int64_t* row_ptr, int32_t* col_idx, int64_t* nnz_out) {
  int64_t cap = oracle_csr_capacity(n, n_pairs);
  uint64_t* keys = (uint64_t*)malloc(sizeof(uint64_t) * (size_t)(cap > 0 ? cap : 1));
  if (!keys) return 1;
  int64_t cnt = 0;
  for (int64_t e = 0; e < n_pairs; ++e) {
    uint64_t s = src[e], d = dst[e];
    if (s == d) continue;                              /* drop self-pairs */
    if (s >= (uint64_t)n || d >= (uint64_t)n) { free(keys); return 2; }
    keys[cnt++] = (s << 32) | d;
    if (flags & 1u) keys[cnt++] = (d << 32) | s;       /* symmetrize (A4) */
  }
  cnt = sort_unique(keys, cnt);                        /* dedup (A3) */
  if (flags & 4u) {                                    /* isolated-vertex fix (A2) */
    char* has = (char*)calloc((size_t)(n > 0 ? n : 1), 1);
    for (int64_t i = 0; i < cnt; ++i) has[keys[i] >> 32] = 1;
    int64_t base = cnt;
    for (int64_t v = 0; v < n; ++v) {
      if (has[v] || n < 2) continue;
      uint64_t u = (uint64_t)((v + 1) % n);
      keys[base++] = ((uint64_t)v << 32) | u;
      keys[base++] = (u << 32) | (uint64_t)v;
    }
    free(has);
    cnt = base;
  }
  if (flags & 2u)                                      /* self-loops (A1) */
    for (int64_t v = 0; v < n; ++v) keys[cnt++] = ((uint64_t)v << 32) | (uint64_t)v;
  cnt = sort_unique(keys, cnt);
  for (int64_t v = 0; v <= n; ++v) row_ptr[v] = 0;
  for (int64_t i = 0; i < cnt; ++i) {
    row_ptr[(keys[i] >> 32) + 1] += 1;
    col_idx[i] = (int32_t)(keys[i] & 0xFFFFFFFFull);
  }
  for (int64_t v = 0; v < n; ++v) row_ptr[v + 1] += row_ptr[v];
  *nnz_out = cnt;
  free(keys);
  return 0;
}

/* Transpose of a CSR pattern: for every column j the list of stored entries
 * (i,j) as positions p into col_idx, ascending in i.  Used for the column
 * sums of the backward pass ("reversed graph").            */
static void build_csc(int64_t n, const int64_t* rp, const int32_t* ci, int64_t* cp, int64_t* pos) {
  int64_t nnz = rp[n];
  for (int64_t j = 0; j <= n; ++j) cp[j] = 0;
  for (int64_t p = 0; p < nnz; ++p) cp[ci[p] + 1] += 1;
  for (int64_t j = 0; j < n; ++j) cp[j + 1] += cp[j];
  int64_t* fill = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n > 0 ? n : 1));
  for (int64_t j = 0; j < n; ++j) fill[j] = cp[j];
  for (int64_t i = 0; i < n; ++i)
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) pos[fill[ci[p]]++] = p;
  free(fill);
}
static int64_t* row_of_edge(int64_t n, const int64_t* rp) {
  int64_t* r = (int64_t*)malloc(sizeof(int64_t) * (size_t)(rp[n] > 0 ? rp[n] : 1));
  for (int64_t i = 0; i < n; ++i)
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) r[p] = i;
  return r;
}

/* dense C[n x c] = A[n x b] * B[b x c] (row-major), the library-primitive MM */
static void mm(int64_t n, int b, int c, const double* A, const double* B, double* C) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    for (int q = 0; q < c; ++q) {
      double acc = 0.0;
      for (int r = 0; r < b; ++r) acc += A[i * b + r] * B[(int64_t)r * c + q];
      C[i * c + q] = acc;
    }
}
/* C[b x c] = A^T B with A[n x b], B[n x c] (reduction over the n rows) */
static void mm_tn(int64_t n, int b, int c, const double* A, const double* B, double* C) {
#pragma omp parallel for schedule(static)
  for (int rq = 0; rq < b * c; ++rq) {
    int r = rq / c, q = rq % c;
    double acc = 0.0;
    for (int64_t i = 0; i < n; ++i) acc += A[i * b + r] * B[i * c + q];
    C[rq] = acc;
  }
}
/* C[n x b] = A[n x c] * B^T with B[b x c] */
static void mm_nt(int64_t n, int c, int b, const double* A, const double* B, double* C) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    for (int r = 0; r < b; ++r) {
      double acc = 0.0;
      for (int q = 0; q < c; ++q) acc += A[i * c + q] * B[(int64_t)r * c + q];
      C[i * b + r] = acc;
    }
}

/* ================================================================== */
/* GAT (PAPER.md:77-79 local formula; :177 global Psi = sm(A (.) sigma(C)),
 * C_ij = s_i + t_j; heads concatenated, reading A10; LeakyReLU(slope),
 * reading A5).  Outputs (all caller-allocated):
 *   P[n x kout] = H W (PAPER.md:141 H' = HW)
 *   s,t[n x heads]: s_i^h = P_i^h . a1^h, t_j^h = P_j^h . a2^h
 *   alpha[nnz x heads], m,l[n x heads] (row max / row sum of exp)
 *   Z[n x kout] = sum_j alpha_ij P_j ; Hout = sigma(Z)                   */
/* BF16 storage mode (north_star "1e-2 with BF16 projection"; DESIGN.md reading
 * B1): the projected rows P and the backward's G are STORED in bfloat16 — the
 * value the kernels gather is round(fp32(x)) to the nearest bf16 (ties to even),
 * exactly what an fp32 result converted with __float2bfloat16_rn holds.        */
static double bf16_round(double x) {
  float f = (float)x;
  uint32_t u;
  memcpy(&u, &f, 4);
  if ((u & 0x7f800000u) != 0x7f800000u) {  /* finite: round to nearest even */
    u += 0x7fffu + ((u >> 16) & 1u);
    u &= 0xffff0000u;
  }
  memcpy(&f, &u, 4);
  return (double)f;
}

/* AGNN / VA BF16 storage mode (reading B2): the gathered operands
 * are the layer input H and the backward's M = G W^T, both stored in bfloat16:
 * the layer computes on H~ = bf16(fp32(H)) throughout (the caller rounds the
 * input with oracle_bf16_round) and M~ = bf16(fp32(M)) replaces M everywhere. */
int oracle_bf16_round(int64_t count, double* x) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < count; ++i) x[i] = bf16_round(x[i]);
  return 0;
}

static int gat_forward_impl(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                            int heads, const double* H, const double* W, const double* a,
                            double slope, int act, double* P, double* s, double* t, double* alpha,
                            double* m, double* l, double* Z, double* Hout, int bf16) {
  if (heads <= 0 || kout % heads) return 1;
  const int d = kout / heads;
  mm(n, k, kout, H, W, P);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i)
    for (int h = 0; h < heads; ++h) {
      double si = 0.0, ti = 0.0;
      for (int c = 0; c < d; ++c) {
        si += P[i * kout + h * d + c] * a[h * 2 * d + c];
        ti += P[i * kout + h * d + c] * a[h * 2 * d + d + c];
      }
      s[i * heads + h] = si;
      t[i * heads + h] = ti;
    }
  /* BF16 mode: the scores above come from the unrounded projection (a' = W a,
   * PAPER.md:141, is its own GEMM column); what is stored and gathered is P~ */
  if (bf16) {
#pragma omp parallel for schedule(static)
    for (int64_t x = 0; x < n * kout; ++x) P[x] = bf16_round(P[x]);
  }
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    for (int h = 0; h < heads; ++h) {
      /* e_ij = sigma(a^T [W h_i || W h_j]) = LReLU(s_i + t_j) */
      double mi = -INFINITY;
      for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
        double pre = s[i * heads + h] + t[(int64_t)ci[p] * heads + h];
        double e = pre > 0.0 ? pre : slope * pre;
        if (e > mi) mi = e;
      }
      double li = 0.0;
      for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
        double pre = s[i * heads + h] + t[(int64_t)ci[p] * heads + h];
        double e = pre > 0.0 ? pre : slope * pre;
        li += exp(e - mi);
      }
      for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
        double pre = s[i * heads + h] + t[(int64_t)ci[p] * heads + h];
        double e = pre > 0.0 ? pre : slope * pre;
        alpha[p * heads + h] = exp(e - mi) / li;
      }
      m[i * heads + h] = rp[i + 1] > rp[i] ? mi : 0.0;
      l[i * heads + h] = li;
      for (int c = 0; c < d; ++c) {
        double z = 0.0;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p)
          z += alpha[p * heads + h] * P[(int64_t)ci[p] * kout + h * d + c];
        Z[i * kout + h * d + c] = z;
      }
    }
    for (int q = 0; q < kout; ++q) Hout[i * kout + q] = act_f(act, Z[i * kout + q]);
  }
  return 0;
}
int oracle_gat_forward(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout, int heads,
                       const double* H, const double* W, const double* a, double slope, int act,
                       double* P, double* s, double* t, double* alpha, double* m, double* l,
                       double* Z, double* Hout) {
  return gat_forward_impl(n, rp, ci, k, kout, heads, H, W, a, slope, act, P, s, t, alpha, m, l, Z,
                          Hout, 0);
}
/* BF16 storage mode: P (output) holds the stored P~ */
int oracle_gat_forward_bf16(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                            int heads, const double* H, const double* W, const double* a,
                            double slope, int act, double* P, double* s, double* t, double* alpha,
                            double* m, double* l, double* Z, double* Hout) {
  return gat_forward_impl(n, rp, ci, k, kout, heads, H, W, a, slope, act, P, s, t, alpha, m, l, Z,
                          Hout, 1);
}

/* GAT backward (Eq. 3-6; derivation in DESIGN.md §2,
 * readings A11 Psi^T, A12 da):
 *   G = dHout (.) sigma'(Z)
 *   delta_i = G_i^h . Z_i^h ; dalpha_ij = G_i^h . P_j^h
 *   dc_ij = alpha_ij (dalpha_ij - delta_i) * (s_i + t_j > 0 ? 1 : slope)
 *   ds_i = sum_j dc_ij ; dt_j = sum_i dc_ij
 *   dP_j^h = sum_i alpha_ij G_i^h + ds_j a1^h + dt_j a2^h
 *   da1^h = sum_i ds_i P_i^h ; da2^h = sum_j dt_j P_j^h
 *   dW = H^T dP ; dH = dP W^T
 * Outputs: dH[n x k], dW[k x kout], da[heads x 2d]; G, dP optional (NULL). */
static int gat_backward_impl(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                             int heads, const double* H, const double* W, const double* a,
                             double slope, int act, const double* P, const double* s,
                             const double* t, const double* alpha, const double* Z,
                             const double* dHout, double* dH, double* dW, double* da,
                             double* G_out, double* dP_out, int bf16) {
  if (heads <= 0 || kout % heads) return 1;
  const int d = kout / heads;
  const int64_t nnz = rp[n];
  double* G = (double*)malloc(sizeof(double) * (size_t)(n * kout + 1));
  double* delta = (double*)malloc(sizeof(double) * (size_t)(n * heads + 1));
  double* dc = (double*)malloc(sizeof(double) * (size_t)(nnz * heads + 1));
  double* ds = (double*)malloc(sizeof(double) * (size_t)(n * heads + 1));
  double* dt = (double*)malloc(sizeof(double) * (size_t)(n * heads + 1));
  double* dP = (double*)malloc(sizeof(double) * (size_t)(n * kout + 1));
  int64_t* cp = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  int64_t* pos = (int64_t*)malloc(sizeof(int64_t) * (size_t)(nnz + 1));
  int64_t* erow = row_of_edge(n, rp);
  build_csc(n, rp, ci, cp, pos);

#pragma omp parallel for schedule(static)
  for (int64_t x = 0; x < n * kout; ++x) {
    G[x] = dHout[x] * act_df(act, Z[x]);
    if (bf16) G[x] = bf16_round(G[x]);  /* BF16 mode: G~ is stored and used throughout */
  }

#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i)
    for (int h = 0; h < heads; ++h) {
      double dl = 0.0;
      for (int c = 0; c < d; ++c) dl += G[i * kout + h * d + c] * Z[i * kout + h * d + c];
      delta[i * heads + h] = dl;
      double dsi = 0.0;
      for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
        int64_t j = ci[p];
        double da_ij = 0.0;
        for (int c = 0; c < d; ++c) da_ij += G[i * kout + h * d + c] * P[j * kout + h * d + c];
        double pre = s[i * heads + h] + t[j * heads + h];
        double lam = pre > 0.0 ? 1.0 : slope;
        dc[p * heads + h] = alpha[p * heads + h] * (da_ij - dl) * lam;
        dsi += dc[p * heads + h];
      }
      ds[i * heads + h] = dsi;
    }

  /* column role over the reversed graph: entries (i,j) of column j */
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t j = 0; j < n; ++j)
    for (int h = 0; h < heads; ++h) {
      double dtj = 0.0;
      for (int64_t q = cp[j]; q < cp[j + 1]; ++q) dtj += dc[pos[q] * heads + h];
      dt[j * heads + h] = dtj;
      for (int c = 0; c < d; ++c) {
        double acc = 0.0;
        for (int64_t q = cp[j]; q < cp[j + 1]; ++q) {
          int64_t p = pos[q], i = erow[p];
          acc += alpha[p * heads + h] * G[i * kout + h * d + c];
        }
        dP[j * kout + h * d + c] =
            acc + ds[j * heads + h] * a[h * 2 * d + c] + dtj * a[h * 2 * d + d + c];
      }
    }

  for (int h = 0; h < heads; ++h)
    for (int c = 0; c < d; ++c) {
      double a1 = 0.0, a2 = 0.0;
      for (int64_t i = 0; i < n; ++i) {
        a1 += ds[i * heads + h] * P[i * kout + h * d + c];
        a2 += dt[i * heads + h] * P[i * kout + h * d + c];
      }
      da[h * 2 * d + c] = a1;
      da[h * 2 * d + d + c] = a2;
    }
  mm_tn(n, k, kout, H, dP, dW);
  if (dH) mm_nt(n, kout, k, dP, W, dH);
  if (G_out) memcpy(G_out, G, sizeof(double) * (size_t)(n * kout));
  if (dP_out) memcpy(dP_out, dP, sizeof(double) * (size_t)(n * kout));
  free(G); free(delta); free(dc); free(ds); free(dt); free(dP); free(cp); free(pos); free(erow);
  return 0;
}
int oracle_gat_backward(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout, int heads,
                        const double* H, const double* W, const double* a, double slope, int act,
                        const double* P, const double* s, const double* t, const double* alpha,
                        const double* Z, const double* dHout, double* dH, double* dW, double* da,
                        double* G_out, double* dP_out) {
  return gat_backward_impl(n, rp, ci, k, kout, heads, H, W, a, slope, act, P, s, t, alpha, Z,
                           dHout, dH, dW, da, G_out, dP_out, 0);
}
/* BF16 storage mode: P is the forward's stored P~; G is rounded to G~ */
int oracle_gat_backward_bf16(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                             int heads, const double* H, const double* W, const double* a,
                             double slope, int act, const double* P, const double* s,
                             const double* t, const double* alpha, const double* Z,
                             const double* dHout, double* dH, double* dW, double* da,
                             double* G_out, double* dP_out) {
  return gat_backward_impl(n, rp, ci, k, kout, heads, H, W, a, slope, act, P, s, t, alpha, Z,
                           dHout, dH, dW, da, G_out, dP_out, 1);
}

/* ================================================================== */
/* AGNN (Psi = A (.) (H_x (/) n n^T), n_i = ||h_i||; reading A8:
 * softmax over each row with temperature beta, nu_i = max(||H_i||, eps)).
 * Aggregate first: X = Psi H, Z = X W, Hout = sigma(Z).
 * Outputs: nu[n], alpha[nnz], m,l[n], X[n x k], Z[n x kout], Hout.       */
int oracle_agnn_forward(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                        const double* H, const double* W, double beta, double eps, int act,
                        double* nu, double* alpha, double* m, double* l, double* X, double* Z,
                        double* Hout) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) {
    double ss = 0.0;
    for (int c = 0; c < k; ++c) ss += H[i * k + c] * H[i * k + c];
    double nrm = sqrt(ss);
    nu[i] = nrm > eps ? nrm : eps;
  }
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    double mi = -INFINITY;
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
      int64_t j = ci[p];
      double dot = 0.0;
      for (int c = 0; c < k; ++c) dot += H[i * k + c] * H[j * k + c];
      double cij = beta * dot / (nu[i] * nu[j]);   /* c_ij = beta H^_i . H^_j */
      alpha[p] = cij;                              /* scores, normalised below */
      if (cij > mi) mi = cij;
    }
    double li = 0.0;
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) li += exp(alpha[p] - mi);
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) alpha[p] = exp(alpha[p] - mi) / li;
    m[i] = rp[i + 1] > rp[i] ? mi : 0.0;
    l[i] = li;
    for (int c = 0; c < k; ++c) {
      double x = 0.0;
      for (int64_t p = rp[i]; p < rp[i + 1]; ++p) x += alpha[p] * H[(int64_t)ci[p] * k + c];
      X[i * k + c] = x;
    }
  }
  mm(n, k, kout, X, W, Z);
#pragma omp parallel for schedule(static)
  for (int64_t x = 0; x < n * kout; ++x) Hout[x] = act_f(act, Z[x]);
  return 0;
}

/* AGNN backward (Eq. 6 with dPsi/dW = 0):
 *   G = dHout (.) sigma'(Z); dW = X^T G; M = G W^T
 *   delta_i = M_i . X_i ; dalpha_ij = M_i . H_j ; dc_ij = beta alpha_ij (dalpha_ij - delta_i)
 *   dH^_j = sum_{(j,i)} dc_ji H^_i + sum_{(i,j)} dc_ij H^_i
 *   dH_j  = sum_{(i,j)} alpha_ij M_i + (dH^_j - (dH^_j . H^_j) H^_j) / nu_j
 *           (nu_j == eps branch: dH^_j / nu_j, nu treated as constant)     */
static int agnn_backward_impl(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                              const double* H, const double* W, double beta, double eps, int act,
                              const double* nu, const double* alpha, const double* X,
                              const double* Z, const double* dHout, double* dH, double* dW,
                              int bf16) {
  const int64_t nnz = rp[n];
  double* G = (double*)malloc(sizeof(double) * (size_t)(n * kout + 1));
  double* M = (double*)malloc(sizeof(double) * (size_t)(n * k + 1));
  double* dc = (double*)malloc(sizeof(double) * (size_t)(nnz + 1));
  int64_t* cp = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  int64_t* pos = (int64_t*)malloc(sizeof(int64_t) * (size_t)(nnz + 1));
  int64_t* erow = row_of_edge(n, rp);
  build_csc(n, rp, ci, cp, pos);
#pragma omp parallel for schedule(static)
  for (int64_t x = 0; x < n * kout; ++x) G[x] = dHout[x] * act_df(act, Z[x]);
  mm_tn(n, k, kout, X, G, dW);
  mm_nt(n, kout, k, G, W, M);
  if (bf16) oracle_bf16_round(n * k, M);  /* BF16 mode (reading B2): M~ used throughout */
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    double dl = 0.0;
    for (int c = 0; c < k; ++c) dl += M[i * k + c] * X[i * k + c];
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
      int64_t j = ci[p];
      double dot = 0.0;
      for (int c = 0; c < k; ++c) dot += M[i * k + c] * H[j * k + c];
      dc[p] = beta * alpha[p] * (dot - dl);
    }
  }
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t j = 0; j < n; ++j) {
    double* dhat = (double*)malloc(sizeof(double) * (size_t)k);
    for (int c = 0; c < k; ++c) dhat[c] = 0.0;
    for (int64_t p = rp[j]; p < rp[j + 1]; ++p) {          /* (j,i): j is the centre */
      int64_t i = ci[p];
      for (int c = 0; c < k; ++c) dhat[c] += dc[p] * H[i * k + c] / nu[i];
    }
    for (int64_t q = cp[j]; q < cp[j + 1]; ++q) {          /* (i,j): i is the centre */
      int64_t p = pos[q], i = erow[p];
      for (int c = 0; c < k; ++c) dhat[c] += dc[p] * H[i * k + c] / nu[i];
    }
    double proj = 0.0;
    for (int c = 0; c < k; ++c) proj += dhat[c] * H[j * k + c] / nu[j];
    const int on_eps = !(nu[j] > eps) ;
    for (int c = 0; c < k; ++c) {
      double acc = 0.0;
      for (int64_t q = cp[j]; q < cp[j + 1]; ++q) {
        int64_t p = pos[q], i = erow[p];
        acc += alpha[p] * M[i * k + c];
      }
      double g = on_eps ? dhat[c] / nu[j] : (dhat[c] - proj * H[j * k + c] / nu[j]) / nu[j];
      dH[j * k + c] = acc + g;
    }
    free(dhat);
  }
  free(G); free(M); free(dc); free(cp); free(pos); free(erow);
  return 0;
}
int oracle_agnn_backward(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                         const double* H, const double* W, double beta, double eps, int act,
                         const double* nu, const double* alpha, const double* X, const double* Z,
                         const double* dHout, double* dH, double* dW) {
  return agnn_backward_impl(n, rp, ci, k, kout, H, W, beta, eps, act, nu, alpha, X, Z, dHout, dH,
                            dW, 0);
}
int oracle_agnn_backward_bf16(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                              const double* H, const double* W, double beta, double eps, int act,
                              const double* nu, const double* alpha, const double* X,
                              const double* Z, const double* dHout, double* dH, double* dW) {
  return agnn_backward_impl(n, rp, ci, k, kout, H, W, beta, eps, act, nu, alpha, X, Z, dHout, dH,
                            dW, 1);
}

/* ================================================================== */
/* VA (PAPER.md:173 Psi = A (.) (H H^T), no softmax; Eq. 7 at :262):
 *   S_ij = A_ij (H_i . H_j); X = S H; Z = X W; Hout = sigma(Z)          */
int oracle_va_forward(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                      const double* H, const double* W, int act, double* S, double* X, double* Z,
                      double* Hout) {
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i) {
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
      int64_t j = ci[p];
      double dot = 0.0;
      for (int c = 0; c < k; ++c) dot += H[i * k + c] * H[j * k + c];
      S[p] = dot;
    }
    for (int c = 0; c < k; ++c) {
      double x = 0.0;
      for (int64_t p = rp[i]; p < rp[i + 1]; ++p) x += S[p] * H[(int64_t)ci[p] * k + c];
      X[i * k + c] = x;
    }
  }
  mm(n, k, kout, X, W, Z);
#pragma omp parallel for schedule(static)
  for (int64_t x = 0; x < n * kout; ++x) Hout[x] = act_f(act, Z[x]);
  return 0;
}

/* VA backward, Eq. 11-13 (reading A11: Psi^T):
 *   G = dHout (.) sigma'(Z); M = G W^T (Eq. 12); N = A (.) (M H^T) (Eq. 12)
 *   Gamma = dH = (N + N^T) H + (A^T (.) H_x) M (Eq. 11)
 *   Y = dW = H^T (A^T (.) H_x) G = X^T G (Eq. 13)                        */
static int va_backward_impl(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                            const double* H, const double* W, int act, const double* S,
                            const double* X, const double* Z, const double* dHout, double* dH,
                            double* dW, int bf16) {
  const int64_t nnz = rp[n];
  double* G = (double*)malloc(sizeof(double) * (size_t)(n * kout + 1));
  double* M = (double*)malloc(sizeof(double) * (size_t)(n * k + 1));
  double* N = (double*)malloc(sizeof(double) * (size_t)(nnz + 1));
  int64_t* cp = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  int64_t* pos = (int64_t*)malloc(sizeof(int64_t) * (size_t)(nnz + 1));
  int64_t* erow = row_of_edge(n, rp);
  build_csc(n, rp, ci, cp, pos);
#pragma omp parallel for schedule(static)
  for (int64_t x = 0; x < n * kout; ++x) G[x] = dHout[x] * act_df(act, Z[x]);
  mm_tn(n, k, kout, X, G, dW);
  mm_nt(n, kout, k, G, W, M);
  if (bf16) oracle_bf16_round(n * k, M);  /* BF16 mode (reading B2): M~ used throughout */
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i)
    for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
      int64_t j = ci[p];
      double dot = 0.0;
      for (int c = 0; c < k; ++c) dot += M[i * k + c] * H[j * k + c];
      N[p] = dot;
    }
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t j = 0; j < n; ++j)
    for (int c = 0; c < k; ++c) {
      double acc = 0.0;
      for (int64_t p = rp[j]; p < rp[j + 1]; ++p)            /* N H        */
        acc += N[p] * H[(int64_t)ci[p] * k + c];
      for (int64_t q = cp[j]; q < cp[j + 1]; ++q) {          /* N^T H, (A^T (.) H_x) M */
        int64_t p = pos[q], i = erow[p];
        acc += N[p] * H[i * k + c] + S[p] * M[i * k + c];
      }
      dH[j * k + c] = acc;
    }
  free(G); free(M); free(N); free(cp); free(pos); free(erow);
  return 0;
}
int oracle_va_backward(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                       const double* H, const double* W, int act, const double* S,
                       const double* X, const double* Z, const double* dHout, double* dH,
                       double* dW) {
  return va_backward_impl(n, rp, ci, k, kout, H, W, act, S, X, Z, dHout, dH, dW, 0);
}
int oracle_va_backward_bf16(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                            const double* H, const double* W, int act, const double* S,
                            const double* X, const double* Z, const double* dHout, double* dH,
                            double* dW) {
  return va_backward_impl(n, rp, ci, k, kout, H, W, act, S, X, Z, dHout, dH, dW, 1);
}

/* ================================================================== */
/* C-GNN layer over a semiring ("C-GNNs ... sigma(A H W) ... the
 * adjacency matrix A (potentially normalized)"; §4.3 the
 * aggregation (+) as a matrix product over a semiring; readings C1-C4 in
 * DESIGN.md §2):
 *   agg 0 SUM   real semiring (R, +, *, 0, 1):      X_i = sum_{j in N(i)} H_j
 *   agg 1 MEAN  averaging semiring (tuples, :201):  X_i = (1/|N(i)|) sum_j H_j
 *   agg 2 GCN   symmetric normalisation of A:       X_i = sum_j H_j / sqrt(d_i d_j)
 *   agg 3 MAX   tropical (R u {-inf}, max, +):      X_ic = max_j H_jc
 *   agg 4 MIN   tropical (R u {+inf}, min, +):      X_ic = min_j H_jc
 * d_i = |N(i)| (stored entries of row i).  Z = X W, Hout = sigma(Z).  An empty
 * row gives X_i = 0 (reading C3).  MAX/MIN record the arg index (the first,
 * i.e. smallest, column j among ties; reading C4) in arg[n x k].          */
static double cg_coef(int agg, const int64_t* rp, int64_t i, int64_t j) {
  const double di = (double)(rp[i + 1] - rp[i]), dj = (double)(rp[j + 1] - rp[j]);
  if (agg == 1) return 1.0 / di;
  if (agg == 2) return 1.0 / sqrt(di * dj);
  return 1.0;
}
int oracle_cgnn_forward(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                        const double* H, const double* W, int agg, int act, double* X,
                        int32_t* arg, double* Z, double* Hout) {
  if (agg < 0 || agg > 4) return 1;
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t i = 0; i < n; ++i)
    for (int c = 0; c < k; ++c) {
      if (agg <= 2) {
        double x = 0.0;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p)
          x += cg_coef(agg, rp, i, ci[p]) * H[(int64_t)ci[p] * k + c];
        X[i * k + c] = x;
      } else {
        int64_t best = -1;
        for (int64_t p = rp[i]; p < rp[i + 1]; ++p) {
          const double v = H[(int64_t)ci[p] * k + c];
          if (best < 0 || (agg == 3 ? v > H[best * k + c] : v < H[best * k + c])) best = ci[p];
        }
        X[i * k + c] = best < 0 ? 0.0 : H[best * k + c];
        arg[i * k + c] = (int32_t)best;
      }
    }
  mm(n, k, kout, X, W, Z);
#pragma omp parallel for schedule(static)
  for (int64_t x = 0; x < n * kout; ++x) Hout[x] = act_f(act, Z[x]);
  return 0;
}

/* Backward: G = dHout (.) sigma'(Z); dW = X^T G; M = G W^T = dL/dX;
 *   SUM/MEAN/GCN: dH_j = sum_{(i,j) stored} coef_ij M_i     (= A'^T M)
 *   MAX/MIN:      dH_jc = sum_{(i,j) stored, arg_ic = j} M_ic              */
int oracle_cgnn_backward(int64_t n, const int64_t* rp, const int32_t* ci, int k, int kout,
                         const double* H, const double* W, int agg, int act, const double* X,
                         const int32_t* arg, const double* Z, const double* dHout, double* dH,
                         double* dW) {
  const int64_t nnz = rp[n];
  (void)H;
  double* G = (double*)malloc(sizeof(double) * (size_t)(n * kout + 1));
  double* M = (double*)malloc(sizeof(double) * (size_t)(n * k + 1));
  int64_t* cp = (int64_t*)malloc(sizeof(int64_t) * (size_t)(n + 1));
  int64_t* pos = (int64_t*)malloc(sizeof(int64_t) * (size_t)(nnz + 1));
  int64_t* erow = row_of_edge(n, rp);
  build_csc(n, rp, ci, cp, pos);
#pragma omp parallel for schedule(static)
  for (int64_t x = 0; x < n * kout; ++x) G[x] = dHout[x] * act_df(act, Z[x]);
  mm_tn(n, k, kout, X, G, dW);
  mm_nt(n, kout, k, G, W, M);
#pragma omp parallel for schedule(dynamic, 64)
  for (int64_t j = 0; j < n; ++j)
    for (int c = 0; c < k; ++c) {
      double acc = 0.0;
      for (int64_t q = cp[j]; q < cp[j + 1]; ++q) {
        const int64_t i = erow[pos[q]];
        if (agg <= 2) acc += cg_coef(agg, rp, i, j) * M[i * k + c];
        else if (arg[i * k + c] == (int32_t)j) acc += M[i * k + c];
      }
      dH[j * k + c] = acc;
    }
  free(G); free(M); free(cp); free(pos); free(erow);
  return 0;
}

/* ================================================================== */
/* 1D row-block partition bounds (reading A20; the paper's own scheme is 2D,
 * PAPER.md:321): w(r) = row_ptr[r] + c_v r ; bounds[0] = 0, bounds[P] = n,
 * bounds[p] = min{ r : w(r) >= ceil(p w(n) / P) }.                       */
int oracle_partition(int64_t n, const int64_t* rp, int world, int64_t c_v, int64_t* bounds) {
  if (world < 1) return 1;
  const int64_t wn = rp[n] + c_v * n;
  bounds[0] = 0;
  bounds[world] = n;
  for (int p = 1; p < world; ++p) {
    int64_t target = (p * wn + world - 1) / world;
    int64_t r = 0;
    while (r < n && rp[r] + c_v * r < target) ++r;
    bounds[p] = r;
  }
  return 0;
}
