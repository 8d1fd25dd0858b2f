// common.cuh — shared device helpers and internal structures of libagnn.so.
#pragma once
#include <vector>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <string>

#include "agnn.h"

namespace agnn {

constexpr float kLog2e = 1.4426950408889634f;
constexpr int kNumSMs = 148;
constexpr int kBundleEdges = 32;  // stored entries per short-row bundle (one warp batch)

// ---- error plumbing (host) -------------------------------------------------
void set_error(const std::string& msg);
agnn_status fail(agnn_status st, const std::string& msg);
agnn_status cuda_status(cudaError_t e, const char* what);
void count_launch(int n = 1);
// live per-kernel timing (agnn_profile_*): an event is recorded on the launch
// stream after every kernel; a kernel's time is the gap to the previous marker.
extern bool g_profiling;
void prof_mark(const char* name, cudaStream_t s);

#define AGNN_CUDA_TRY(expr)                                            \
  do {                                                                 \
    cudaError_t _e = (expr);                                           \
    if (_e != cudaSuccess) return ::agnn::cuda_status(_e, #expr);      \
  } while (0)

// (expects the launch stream in a variable named `s`)
#define AGNN_LAUNCH_CHECK(name)                                        \
  do {                                                                 \
    ::agnn::count_launch();                                            \
    cudaError_t _e = cudaGetLastError();                               \
    if (_e != cudaSuccess) return ::agnn::cuda_status(_e, name);       \
    if (::agnn::g_profiling) ::agnn::prof_mark(name, s);               \
  } while (0)

// ---- device helpers ----------------------------------------------------------
__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

__device__ __forceinline__ float4 ldg4(const float* p) {
  return __ldg(reinterpret_cast<const float4*>(p));
}
// streaming (read-once) load: do not allocate in L1
__device__ __forceinline__ float4 ld_stream4(const float* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p));
  return r;
}
__device__ __forceinline__ void st4(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }

// ---- L2 residency of gathered rows (plan column classes, see plan.cu) ----------
// A gathered neighbour row is loaded with an explicit L2 eviction policy: rows of
// the most-gathered vertices (the hubs of a skewed graph) with evict_last, so they
// stay in the 126 MB L2 across the pass, the rest with evict_first (or normal).
struct L2Pol {
  uint64_t hot, cold;
};
__device__ __forceinline__ L2Pol make_l2pol(int cold_first) {
  L2Pol p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p.hot));
  if (cold_first)
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p.cold));
  else
    asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p.cold));
  return p;
}
__device__ __forceinline__ float4 ldg4_pol(const float* p, uint64_t pol) {
  float4 r;
  asm("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
               : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ uint2 ldg8_pol(const void* p, uint64_t pol) {
  uint2 r;
  asm("ld.global.nc.L2::cache_hint.v2.u32 {%0,%1}, [%2], %3;"
               : "=r"(r.x), "=r"(r.y)
               : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ uint4 ldg16_pol(const void* p, uint64_t pol) {
  uint4 r;
  asm("ld.global.nc.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
               : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ float ldg1_pol(const float* p, uint64_t pol) {
  float r;
  asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(r) : "l"(p), "l"(pol));
  return r;
}

// ---- bfloat16 feature storage (GAT BF16 mode, reading B1) ---------------------
// 4 consecutive bf16 features = 8 bytes; widened to fp32 exactly (bf16 is the high
// half of an fp32), narrowed with round-to-nearest-even (cvt.rn.bf16x2.f32).
typedef __nv_bfloat16 bf16;
__device__ __forceinline__ float4 bf4_to_f4(uint2 u) {
  return make_float4(__uint_as_float(u.x << 16), __uint_as_float(u.x & 0xffff0000u),
                     __uint_as_float(u.y << 16), __uint_as_float(u.y & 0xffff0000u));
}
__device__ __forceinline__ float4 ldg4(const bf16* p) {
  return bf4_to_f4(__ldg(reinterpret_cast<const uint2*>(p)));
}
__device__ __forceinline__ uint32_t pack_bf2(float lo, float hi) {
  uint32_t r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
  return r;
}
__device__ __forceinline__ uint2 f4_to_bf4(float4 v) {
  return make_uint2(pack_bf2(v.x, v.y), pack_bf2(v.z, v.w));
}
__device__ __forceinline__ void st4(bf16* p, float4 v) {
  *reinterpret_cast<uint2*>(p) = f4_to_bf4(v);
}
// the value a bf16 store of v holds, widened back (G~ of reading B1)
__device__ __forceinline__ float4 round_bf4(float4 v) { return bf4_to_f4(f4_to_bf4(v)); }

// a gathered 4-column slice of a feature row as loaded (raw) and widened to fp32:
// bf16 slices stay packed (2 registers) until their use, so twice as many rows
// can be in flight per lane for the same registers
template <typename TP>
struct Slice;
template <>
struct Slice<float> {
  using raw = float4;
  __device__ static __forceinline__ raw load(const float* p) { return ldg4(p); }
  __device__ static __forceinline__ raw load(const float* p, uint64_t pol) {
    return ldg4_pol(p, pol);
  }
  __device__ static __forceinline__ float4 f(raw r) { return r; }
  __device__ static __forceinline__ raw zero() { return make_float4(0.f, 0.f, 0.f, 0.f); }
};
template <>
struct Slice<bf16> {
  using raw = uint2;
  __device__ static __forceinline__ raw load(const bf16* p) {
    return __ldg(reinterpret_cast<const uint2*>(p));
  }
  __device__ static __forceinline__ raw load(const bf16* p, uint64_t pol) { return ldg8_pol(p, pol); }
  __device__ static __forceinline__ float4 f(raw r) { return bf4_to_f4(r); }
  __device__ static __forceinline__ raw zero() { return make_uint2(0u, 0u); }
};


__device__ __forceinline__ float dot4(float4 a, float4 b) {
  return fmaf(a.x, b.x, fmaf(a.y, b.y, fmaf(a.z, b.z, a.w * b.w)));
}
__device__ __forceinline__ float4 f4(float v) { return make_float4(v, v, v, v); }
__device__ __forceinline__ float4 fma4(float s, float4 x, float4 y) {  // s*x + y
  return make_float4(fmaf(s, x.x, y.x), fmaf(s, x.y, y.y), fmaf(s, x.z, y.z), fmaf(s, x.w, y.w));
}
__device__ __forceinline__ float4 mul4(float s, float4 x) {
  return make_float4(s * x.x, s * x.y, s * x.z, s * x.w);
}
__device__ __forceinline__ float4 add4(float4 a, float4 b) {
  return make_float4(a.x + b.x, a.y + b.y, a.z + b.z, a.w + b.w);
}

__device__ __forceinline__ float act_fwd(int act, float z) {
  if (act == AGNN_ACT_RELU) return z > 0.f ? z : 0.f;
  if (act == AGNN_ACT_ELU) return z > 0.f ? z : expm1f(z);
  return z;
}
__device__ __forceinline__ float act_grad(int act, float z) {
  if (act == AGNN_ACT_RELU) return z > 0.f ? 1.f : 0.f;
  if (act == AGNN_ACT_ELU) return z > 0.f ? 1.f : expf(z);
  return 1.f;
}
__device__ __forceinline__ float4 act_fwd4(int act, float4 z) {
  return make_float4(act_fwd(act, z.x), act_fwd(act, z.y), act_fwd(act, z.z), act_fwd(act, z.w));
}

// ---- lane layout of one feature row over a group of lanes -------------------
// A row of K fp32 features is held by LANES lanes, VPL float4 each; the v-th
// float4 of lane q covers columns c = v*LANES*4 + q*4 .. +3 (coalesced).
template <int K, int NH>
struct RowLayout {
  static_assert(K % 16 == 0 && K >= 16 && K <= 256, "K must be 16..256, multiple of 16");
  static constexpr int LANES = (K / 4 >= 32) ? 32 : K / 4;
  static constexpr int VPL = K / (4 * LANES);
  static constexpr int GROUPS = 32 / LANES;
  static constexpr int D = K / NH;  // head width
  static_assert(K % NH == 0 && D % 4 == 0, "head width must be a multiple of 4");
  // lanes sharing one head inside one float4 slot
  static constexpr int HL = (D / 4 < LANES) ? D / 4 : LANES;
  // consecutive v slots spanned by one head (D > 4*LANES)
  static constexpr int VS = (D > 4 * LANES) ? D / (4 * LANES) : 1;
  __device__ static __forceinline__ int col(int v, int q) { return v * LANES * 4 + q * 4; }
  __device__ static __forceinline__ int head(int v, int q) { return col(v, q) / D; }
  // sum x over the lanes of one head (xor butterfly inside aligned HL groups)
  __device__ static __forceinline__ float head_sum(float x) {
#pragma unroll
    for (int o = HL / 2; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    return x;
  }
  // per-slot partial dot products -> full per-head dot product in every slot
  __device__ static __forceinline__ void head_reduce(float (&x)[VPL]) {
    if constexpr (VS > 1) {
#pragma unroll
      for (int v0 = 0; v0 < VPL; v0 += VS) {
        float t = 0.f;
#pragma unroll
        for (int v = 0; v < VS; ++v) t += x[v0 + v];
#pragma unroll
        for (int v = 0; v < VS; ++v) x[v0 + v] = t;
      }
    }
#pragma unroll
    for (int v = 0; v < VPL; ++v) x[v] = head_sum(x[v]);
  }
};

// ---- plan / model (host structures) ------------------------------------------
constexpr int kMaxPeers = 8;

struct Plan {
  int64_t n = 0, row_begin = 0, row_end = 0, n_local = 0, nnz = 0;
  const int64_t* row_ptr = nullptr;   // caller-owned, local rows
  const int32_t* col_idx = nullptr;   // caller-owned
  uint32_t flags = 0;
  int64_t max_deg = 0;
  // work lists (device, plan-owned)
  int chunk = 2048;
  int64_t n_light = 0, n_heavy = 0, n_chunks = 0;
  int32_t* light_rows = nullptr;      // [n_light]
  int32_t* chunk_row = nullptr;       // [n_chunks]
  int32_t* chunk_idx = nullptr;       // [n_chunks] chunk ordinal within its row
  int32_t* heavy_rows = nullptr;      // [n_heavy]
  int32_t* heavy_off = nullptr;       // [n_heavy+1] chunk ranges
  void* meta_block = nullptr;         // single allocation backing the lists
  // light rows split by degree for the short-row kernels (gat_short.cu):
  // short = degree <= short_max, long = the other light rows (both ascending)
  int short_max = 32;
  int64_t n_short = 0, n_long = 0;
  int32_t* short_rows = nullptr;
  int32_t* long_rows = nullptr;
  int4* short_meta = nullptr;         // [n_short] {row, degree, beg lo, beg hi}: one 16-B load;
                                      // the n_short_nz non-empty rows first
  int64_t n_short_nz = 0;
  int4* bundles = nullptr;            // [n_bundles] {first short record, rows, entries, 0}
  int64_t n_bundles = 0;
  void* short_block = nullptr;        // backs short_meta
  int32_t* empty_rows = nullptr;      // [n_empty] local rows without stored entries
  int64_t n_empty = 0;
  // L2 residency classes of the gathered rows (plan.cu "column classes"): a
  // plan-owned copy of col_idx whose bits [hint_shift, 31) hold the class c of
  // the column (c >= q: among the ~2^(21 - (q-1)/4) most-gathered vertices of
  // this rank); null when n > 2^28 or disabled (AGNN_L2_HOT_MB=0)
  int32_t* col_hint = nullptr;
  int hint_shift = 0;
  int n_classes = 0;                  // classes 1..n_classes-1 in use
  int64_t class_rows[64] = {};        // [q] = vertices of class >= q (host)
  // directed patterns (world == 1): the transposed pattern (CSC of the local
  // matrix) and its work lists, for the column role of the backward
  // (PAPER.md:252 Psi^T; reading A4).  Plan-owned; null for symmetric plans.
  int64_t* csc_ptr = nullptr;         // [n+1] column j lists rows i with stored (i,j)
  int32_t* csc_idx = nullptr;         // [nnz]
  int64_t c_light = 0, c_heavy = 0, c_chunks = 0;
  int32_t* c_light_rows = nullptr;
  int32_t* c_chunk_row = nullptr;
  int32_t* c_chunk_idx = nullptr;
  int32_t* c_heavy_rows = nullptr;
  int32_t* c_heavy_off = nullptr;
  void* csc_block = nullptr;          // backs csc_ptr / csc_idx
  void* c_meta_block = nullptr;       // backs the column work lists
  bool directed() const { return !(flags & 1u); }
  // work-decomposition options (agnn_plan_options; include/agnn.h)
  int gat_factored = 1;               // 0 never, 1 k' = 128 only, 2 every width
  int bundle_mode = 1;                // short-row bundles: 0 never, 1 fp32, 2 fp32 + bf16
  int64_t l2_hot_mb = 96;             // evict_last budget; 0: no column classes
  int spmmm = 0;                      // AGNN/VA k = 128 forward: fused SpMMM kernel
  int64_t max_chunks() const { return n_chunks > c_chunks ? n_chunks : c_chunks; }
  // distribution
  int rank = 0, world = 1;
  int64_t* bounds = nullptr;          // host [world+1]
  void* nccl = nullptr;               // ncclComm_t (NCCL exchange)
  // peer-memory exchange (world > 1 without an NCCL id): every rank's replicated
  // buffers and control block are mapped into every other rank (CUDA IPC over
  // NVLink / NVSwitch); see comm.cu
  bool peer = false;
  bool peer_ready = false;
  void* ctl = nullptr;                // plan-owned: barrier flags + reduce slots
  void* peer_ctl[kMaxPeers] = {};     // every rank's control block ([rank] = ctl)
  struct Reg {                        // registered (symmetric) buffer
    char* local;
    size_t bytes;
    char* peer[kMaxPeers];
  };
  std::vector<Reg>* regs = nullptr;
  std::vector<void*>* opened = nullptr;  // IPC mappings to close at destroy
  // needed-rows exchange (comm.cu): the rows of this rank's block that each peer's
  // rows reference (sent by every all-gather instead of the whole block)
  size_t want_off = 0;                // byte offset of this rank's wanted lists in ctl
  int64_t n_wanted = 0;               // columns of other blocks this rank's rows reference
  int32_t* send_idx = nullptr;        // device, plan-owned: rows to push, by peer
  uint8_t* send_mask = nullptr;       // device [n_local]: bit pi = compact peer pi needs the row
  int64_t send_off[kMaxPeers + 1] = {};  // host: peer q's rows are send_idx[send_off[q] ..)
  mutable int64_t epoch = 0;          // barrier generation (host, in stream order)
  mutable int64_t red_calls = 0;      // all-reduce slot-set parity
};

struct Model {
  Plan* plan = nullptr;
  int n_layers = 0;
  agnn_layer_desc* descs = nullptr;
};

// byte layout helpers (aligned sub-buffers inside saved / workspace)
struct Carver {
  char* base;
  size_t off = 0;
  explicit Carver(void* b) : base(static_cast<char*>(b)) {}
  template <typename T>
  T* take(size_t count) {
    off = (off + 255) & ~size_t(255);
    T* p = base ? reinterpret_cast<T*>(base + off) : nullptr;
    off += count * sizeof(T);
    return p;
  }
};

}  // namespace agnn
