// api.cu — the extern "C" surface of libagnn.so (declared in include/agnn.h).
#include <atomic>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <unordered_map>
#include <vector>

#include "internal.cuh"

namespace agnn {

static thread_local std::string g_last_error;
static std::atomic<uint64_t> g_launches{0};

void set_error(const std::string& msg) { g_last_error = msg; }
agnn_status fail(agnn_status st, const std::string& msg) {
  set_error(msg);
  return st;
}
agnn_status cuda_status(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return AGNN_OK;
  return fail(AGNN_ECUDA, std::string(what) + ": " + cudaGetErrorString(e));
}
void count_launch(int n) { g_launches.fetch_add((uint64_t)n, std::memory_order_relaxed); }

// ---- live kernel timing ------------------------------------------------------
bool g_profiling = false;
namespace {
struct Mark {
  std::string name;
  cudaEvent_t prev, ev;
};
std::mutex g_prof_mu;
std::vector<cudaEvent_t> g_ev_pool;
std::vector<Mark> g_marks;
std::unordered_map<cudaStream_t, cudaEvent_t> g_last;
struct Stat {
  double ms = 0;
  long count = 0;
};
std::map<std::string, Stat> g_stats;
cudaEvent_t take_event() {
  if (!g_ev_pool.empty()) {
    cudaEvent_t e = g_ev_pool.back();
    g_ev_pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  cudaEventCreate(&e);
  return e;
}
void drain_marks() {  // caller holds the lock; synchronises on the recorded events
  for (auto& m : g_marks) {
    cudaEventSynchronize(m.ev);
    if (m.prev && !m.name.empty()) {
      float ms = 0;
      if (cudaEventElapsedTime(&ms, m.prev, m.ev) == cudaSuccess) {
        g_stats[m.name].ms += ms;
        g_stats[m.name].count += 1;
      }
    }
  }
  // every event except the latest marker of each stream returns to the pool
  std::vector<cudaEvent_t> keep;
  for (auto& kv : g_last) keep.push_back(kv.second);
  for (auto& m : g_marks) {
    bool k = false;
    for (auto e : keep) k = k || (e == m.ev);
    if (!k) g_ev_pool.push_back(m.ev);
  }
  g_marks.clear();
}
}  // namespace

void prof_mark(const char* name, cudaStream_t s) {
  std::lock_guard<std::mutex> lock(g_prof_mu);
  cudaEvent_t e = take_event();
  cudaEventRecord(e, s);
  auto it = g_last.find(s);
  cudaEvent_t prev = it == g_last.end() ? nullptr : it->second;
  g_marks.push_back(Mark{name ? name : "", prev, e});
  g_last[s] = e;
  if (g_marks.size() > 4096) drain_marks();
}

agnn_status plan_build(Plan& p, cudaStream_t s);
agnn_status plan_options(Plan& p, const agnn_plan_options* o);

// widths with a sparse-kernel instantiation (the dispatch tables of gat.cu,
// agnn_va.cu, cgnn.cu): anything else is rejected here, before any launch
static bool pow2_width(int k) { return k == 16 || k == 32 || k == 64 || k == 128 || k == 256; }
static bool gat_width(int k, int h) {
  if (k == 16) return h == 1 || h == 2 || h == 4;
  return pow2_width(k) && (h == 1 || h == 2 || h == 4 || h == 8);
}

static agnn_status check_desc(const agnn_layer_desc& d) {
  if (d.k_in <= 0 || d.k_out <= 0 || d.k_in % 4 || d.k_out % 4)
    return fail(AGNN_EINVAL, "layer desc: k_in/k_out must be positive multiples of 4");
  if (d.act < AGNN_ACT_NONE || d.act > AGNN_ACT_ELU) return fail(AGNN_EINVAL, "layer desc: act");
  if (d.prec < AGNN_PREC_FP32 || d.prec > AGNN_PREC_BF16) return fail(AGNN_EINVAL, "layer desc: prec");
  if (d.prec == AGNN_PREC_BF16 &&
      !(d.kind == AGNN_GAT && d.k_out == 128 &&
        (d.heads == 1 || d.heads == 2 || d.heads == 4 || d.heads == 8)) &&
      !((d.kind == AGNN_AGNN || d.kind == AGNN_VA) && (d.k_in == 128 || d.k_in == 256)))
    return fail(AGNN_EUNSUPPORTED,
                "AGNN_PREC_BF16: GAT with k_out = 128 and 1/2/4/8 heads, or AGNN / VA with "
                "k_in = 128 / 256");
  if (d.kind == AGNN_GAT) {
    if (d.heads <= 0 || d.k_out % d.heads || (d.k_out / d.heads) % 4)
      return fail(AGNN_EINVAL, "GAT: k_out must split into heads of a multiple of 4 features");
    if (!gat_width(d.k_out, d.heads))
      return fail(AGNN_EUNSUPPORTED,
                  "GAT: (k_out, heads) must be k_out in 16/32/64/128/256 with 1/2/4/8 heads "
                  "(k_out = 16: 1/2/4)");
  } else if (d.kind == AGNN_AGNN || d.kind == AGNN_VA) {
    if (d.heads != 1) return fail(AGNN_EINVAL, "AGNN/VA: heads must be 1");
    if (!pow2_width(d.k_in))
      return fail(AGNN_EUNSUPPORTED, "AGNN/VA: k_in must be 16/32/64/128/256");
  } else if (d.kind == AGNN_CGNN) {
    if (d.heads != 1) return fail(AGNN_EINVAL, "C-GNN: heads must be 1");
    if (d.agg < AGNN_AGG_SUM || d.agg > AGNN_AGG_MIN) return fail(AGNN_EINVAL, "C-GNN: agg");
    if (!pow2_width(d.k_in))
      return fail(AGNN_EUNSUPPORTED, "C-GNN: k_in must be 16/32/64/128/256");
  } else {
    return fail(AGNN_EINVAL, "layer desc: kind");
  }
  return AGNN_OK;
}

static GatShape gat_shape(const agnn_layer_desc& d) {
  return GatShape{d.k_in, d.k_out, d.heads, d.negative_slope, (int)d.act,
                  d.prec == AGNN_PREC_BF16};
}

// C-GNN entry points live in cgnn.cu
agnn_status cg_saved_bytes(const Plan& p, const agnn_layer_desc& d, size_t* b);
agnn_status cg_workspace_bytes(const Plan& p, const agnn_layer_desc& d, size_t* b);
agnn_status cg_forward(const Plan& p, const agnn_layer_desc& d, const float* W, const float* H_in,
                       float* H_out, void* saved, void* ws, cudaStream_t s);
agnn_status cg_backward(const Plan& p, const agnn_layer_desc& d, const float* W,
                        const float* H_in, const void* saved, const float* dH_out, float* dH_in,
                        float* dW, void* ws, cudaStream_t s);

// AGNN / VA entry points live in agnn_va.cu
agnn_status av_saved_bytes(const Plan& p, const agnn_layer_desc& d, size_t* b);
agnn_status av_workspace_bytes(const Plan& p, const agnn_layer_desc& d, size_t* b);
agnn_status av_forward(const Plan& p, const agnn_layer_desc& d, const float* W, const float* H_in,
                       float* H_out, void* saved, void* ws, cudaStream_t s);
agnn_status av_backward(const Plan& p, const agnn_layer_desc& d, const float* W,
                        const float* H_in, const void* saved, const float* dH_out, float* dH_in,
                        float* dW, void* ws, cudaStream_t s);
agnn_status av_debug_attention(const Plan& p, const agnn_layer_desc& d, const void* saved,
                               const float* H_in_full, const int64_t* pos, int64_t count,
                               float* out, cudaStream_t s);

static bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

}  // namespace agnn

using namespace agnn;

struct agnn_plan_s {
  Plan p;
};
struct agnn_model_s {
  Model m;
};

extern "C" {

const char* agnn_status_string(agnn_status s) {
  switch (s) {
    case AGNN_OK: return "AGNN_OK";
    case AGNN_EINVAL: return "AGNN_EINVAL";
    case AGNN_ECUDA: return "AGNN_ECUDA";
    case AGNN_ENCCL: return "AGNN_ENCCL";
    case AGNN_ENOMEM: return "AGNN_ENOMEM";
    case AGNN_EUNSUPPORTED: return "AGNN_EUNSUPPORTED";
    case AGNN_ESTATE: return "AGNN_ESTATE";
  }
  return "AGNN_UNKNOWN";
}

const char* agnn_last_error(void) { return g_last_error.c_str(); }

uint64_t agnn_launch_count(void) { return g_launches.load(); }

agnn_status agnn_debug_gemm_tn(const float* A, int64_t M, int K1, const float* B, int N,
                               float* C, float* ws, cudaStream_t s) {
  if (!A || !B || !C || !ws || M < 0 || K1 <= 0 || N <= 0)
    return fail(AGNN_EINVAL, "agnn_debug_gemm_tn: bad arguments");
  return gemm_tn(A, M, K1, B, N, C, ws, s);
}

size_t agnn_debug_gemm_tn_ws_bytes(int K1, int N) { return gemm_tn_ws_floats(K1, N) * sizeof(float); }

agnn_status agnn_debug_gemm(const float* A, int64_t M, int K, const float* B, int N, float* C,
                            cudaStream_t s) {
  if (!A || !B || !C || M < 0 || K <= 0 || N <= 0)
    return fail(AGNN_EINVAL, "agnn_debug_gemm: bad arguments");
  return gemm_rows(A, M, K, B, true, N, C, N, nullptr, s);
}

agnn_status agnn_profile_enable(int on) {
  std::lock_guard<std::mutex> lock(g_prof_mu);
  g_profiling = on != 0;
  g_last.clear();  // the next call on each stream starts a fresh chain
  return AGNN_OK;
}

agnn_status agnn_profile_report(char* buf, size_t len) {
  std::lock_guard<std::mutex> lock(g_prof_mu);
  drain_marks();
  std::string out;
  for (auto& kv : g_stats) {
    char line[256];
    snprintf(line, sizeof(line), "%s %ld %.6f\n", kv.first.c_str(), kv.second.count, kv.second.ms);
    out += line;
  }
  if (buf && len) {
    strncpy(buf, out.c_str(), len - 1);
    buf[len - 1] = 0;
  }
  return out.size() < len ? AGNN_OK : AGNN_EINVAL;
}

agnn_status agnn_profile_reset(void) {
  std::lock_guard<std::mutex> lock(g_prof_mu);
  drain_marks();
  g_stats.clear();
  g_last.clear();
  return AGNN_OK;
}

agnn_status agnn_plan_create(const agnn_csr* csr, const agnn_dist* dist, cudaStream_t s,
                             agnn_plan_t* out) {
  return agnn_plan_create_ex(csr, dist, nullptr, s, out);
}

agnn_status agnn_plan_create_ex(const agnn_csr* csr, const agnn_dist* dist,
                                const agnn_plan_options* opts, cudaStream_t s, agnn_plan_t* out) {
  try {
    if (!csr || !out) return fail(AGNN_EINVAL, "agnn_plan_create: NULL argument");
    if (csr->n <= 0 || csr->n > INT32_MAX || csr->row_begin < 0 || csr->row_end > csr->n ||
        csr->row_end < csr->row_begin || !csr->row_ptr)
      return fail(AGNN_EINVAL, "agnn_plan_create: bad CSR header (n, row range, row_ptr)");
    if (!(dist && dist->world > 1) && (csr->row_begin != 0 || csr->row_end != csr->n))
      return fail(AGNN_EINVAL,
                  "agnn_plan_create: with world == 1 the CSR must hold every row "
                  "(row_begin == 0, row_end == n)");
    if (csr->flags & ~(uint32_t)(AGNN_CSR_SYMMETRIC | AGNN_PLAN_VERIFY_SYMMETRY))
      return fail(AGNN_EINVAL, "agnn_plan_create: unknown CSR flags");
    auto* h = new (std::nothrow) agnn_plan_s();
    if (!h) return fail(AGNN_ENOMEM, "agnn_plan_create: out of host memory");
    Plan& p = h->p;
    p.n = csr->n;
    p.row_begin = csr->row_begin;
    p.row_end = csr->row_end;
    p.n_local = csr->row_end - csr->row_begin;
    p.row_ptr = csr->row_ptr;
    p.col_idx = csr->col_idx;
    p.flags = csr->flags;
    if (dist && dist->world > 1) {
      if (!dist->bounds || dist->rank < 0 || dist->rank >= dist->world ||
          (!dist->nccl_unique_id && dist->world > kMaxPeers)) {
        delete h;
        return fail(AGNN_EINVAL, "agnn_plan_create: bad dist (unique id / bounds / rank)");
      }
      p.rank = dist->rank;
      p.world = dist->world;
      p.bounds = new int64_t[dist->world + 1];
      memcpy(p.bounds, dist->bounds, sizeof(int64_t) * (dist->world + 1));
      if (p.bounds[0] != 0 || p.bounds[p.world] != p.n || p.bounds[p.rank] != p.row_begin ||
          p.bounds[p.rank + 1] != p.row_end) {
        delete[] p.bounds;
        delete h;
        return fail(AGNN_EINVAL, "agnn_plan_create: bounds do not match the CSR row range");
      }
    }
    agnn_status st = plan_options(p, opts);
    if (st == AGNN_OK) st = plan_build(p, s);
    if (st == AGNN_OK && p.world > 1) st = comm_init(p, dist->nccl_unique_id);
    if (st != AGNN_OK) {
      comm_destroy(p);
      if (p.meta_block) cudaFree(p.meta_block);
      if (p.csc_block) cudaFree(p.csc_block);
      if (p.c_meta_block) cudaFree(p.c_meta_block);
      if (p.short_block) cudaFree(p.short_block);
      if (p.col_hint) cudaFree(p.col_hint);
      delete[] p.bounds;
      delete h;
      return st;
    }
    *out = h;
    return AGNN_OK;
  } catch (const std::exception& e) {
    return fail(AGNN_ENOMEM, std::string("agnn_plan_create: ") + e.what());
  }
}

agnn_status agnn_plan_destroy(agnn_plan_t h) {
  if (!h) return AGNN_OK;
  comm_destroy(h->p);
  if (h->p.meta_block) cudaFree(h->p.meta_block);
  if (h->p.csc_block) cudaFree(h->p.csc_block);
  if (h->p.c_meta_block) cudaFree(h->p.c_meta_block);
  if (h->p.short_block) cudaFree(h->p.short_block);
  if (h->p.col_hint) cudaFree(h->p.col_hint);
  delete[] h->p.bounds;
  delete h;
  return AGNN_OK;
}

agnn_status agnn_plan_info(agnn_plan_t h, int64_t* info) {
  if (!h || !info) return fail(AGNN_EINVAL, "agnn_plan_info: NULL argument");
  const Plan& p = h->p;
  info[0] = p.n_local;
  info[1] = p.nnz;
  info[2] = p.n_light;
  info[3] = p.n_heavy;
  info[4] = p.n_chunks;
  info[5] = p.chunk;
  info[6] = p.max_deg;
  info[7] = p.n;
  info[8] = p.n_short;
  info[9] = p.short_max;
  info[10] = p.n_wanted;
  info[11] = p.send_off[p.world > 1 ? p.world : 0];
  return AGNN_OK;
}

agnn_status agnn_plan_ctl_export(agnn_plan_t h, void* handle, int64_t* offset) {
  if (!h || !handle || !offset) return fail(AGNN_EINVAL, "agnn_plan_ctl_export: NULL argument");
  if (!h->p.peer) return fail(AGNN_ESTATE, "agnn_plan_ctl_export: plan does not use peer exchange");
  return agnn_ipc_export(h->p.ctl, handle, offset);
}

agnn_status agnn_plan_connect(agnn_plan_t h, const void* handles, const int64_t* offsets) {
  if (!h || !handles || !offsets) return fail(AGNN_EINVAL, "agnn_plan_connect: NULL argument");
  Plan& p = h->p;
  if (!p.peer) return fail(AGNN_ESTATE, "agnn_plan_connect: plan does not use peer exchange");
  char* out[kMaxPeers] = {};
  agnn_status st = peer_open(p, handles, offsets, p.ctl, out);
  if (st != AGNN_OK) return st;
  for (int r = 0; r < p.world; ++r) p.peer_ctl[r] = out[r];
  if ((st = peer_send_lists(p)) != AGNN_OK) return st;
  p.peer_ready = true;
  return AGNN_OK;
}

agnn_status agnn_plan_register(agnn_plan_t h, void* local, size_t bytes, const void* handles,
                               const int64_t* offsets) {
  if (!h || !local || !handles || !offsets) return fail(AGNN_EINVAL, "agnn_plan_register: NULL argument");
  Plan& p = h->p;
  if (!p.peer) return fail(AGNN_ESTATE, "agnn_plan_register: plan does not use peer exchange");
  Plan::Reg g;
  g.local = static_cast<char*>(local);
  g.bytes = bytes;
  agnn_status st = peer_open(p, handles, offsets, local, g.peer);
  if (st != AGNN_OK) return st;
  p.regs->push_back(g);
  return AGNN_OK;
}

agnn_status agnn_plan_csc(agnn_plan_t h, int64_t* col_ptr, int32_t* row_idx, int64_t* perm,
                          cudaStream_t s) {
  if (!h || !col_ptr || !row_idx) return fail(AGNN_EINVAL, "agnn_plan_csc: NULL argument");
  const Plan& p = h->p;
  if (p.world != 1 || p.row_begin != 0 || p.n_local != p.n)
    return fail(AGNN_EUNSUPPORTED, "agnn_plan_csc: needs world == 1 and every row in the plan");
  try {
    return build_csc(p.row_ptr, p.col_idx, p.n_local, p.n, p.nnz, col_ptr, row_idx, perm, s);
  } catch (const std::exception& e) {
    return fail(AGNN_ENOMEM, std::string("agnn_plan_csc: ") + e.what());
  }
}

agnn_status agnn_model_create(agnn_plan_t plan, int n_layers, const agnn_layer_desc* descs,
                              agnn_model_t* out) {
  if (!plan || n_layers <= 0 || !descs || !out)
    return fail(AGNN_EINVAL, "agnn_model_create: bad arguments");
  for (int l = 0; l < n_layers; ++l) {
    agnn_status st = check_desc(descs[l]);
    if (st != AGNN_OK) return st;
    if (l > 0 && descs[l].k_in != descs[l - 1].k_out)
      return fail(AGNN_EINVAL, "agnn_model_create: k_in of a layer must equal k_out of the previous");
  }
  auto* h = new (std::nothrow) agnn_model_s();
  if (!h) return fail(AGNN_ENOMEM, "agnn_model_create: out of host memory");
  h->m.plan = &plan->p;
  h->m.n_layers = n_layers;
  h->m.descs = new agnn_layer_desc[n_layers];
  memcpy(h->m.descs, descs, sizeof(agnn_layer_desc) * n_layers);
  *out = h;
  return AGNN_OK;
}

agnn_status agnn_model_destroy(agnn_model_t h) {
  if (!h) return AGNN_OK;
  delete[] h->m.descs;
  delete h;
  return AGNN_OK;
}

static agnn_status layer_of(agnn_model_t h, int layer, const agnn_layer_desc** d) {
  if (!h) return fail(AGNN_EINVAL, "NULL model");
  if (layer < 0 || layer >= h->m.n_layers) return fail(AGNN_EINVAL, "layer index out of range");
  *d = &h->m.descs[layer];
  return AGNN_OK;
}

agnn_status agnn_saved_bytes(agnn_model_t h, int layer, size_t* bytes) {
  const agnn_layer_desc* d;
  agnn_status st = layer_of(h, layer, &d);
  if (st != AGNN_OK) return st;
  if (!bytes) return fail(AGNN_EINVAL, "agnn_saved_bytes: NULL");
  if (d->kind == AGNN_GAT) {
    *bytes = gat_saved_bytes(*h->m.plan, gat_shape(*d));
    return AGNN_OK;
  }
  if (d->kind == AGNN_CGNN) return cg_saved_bytes(*h->m.plan, *d, bytes);
  return av_saved_bytes(*h->m.plan, *d, bytes);
}

agnn_status agnn_workspace_bytes(agnn_model_t h, int layer, size_t* bytes) {
  const agnn_layer_desc* d;
  agnn_status st = layer_of(h, layer, &d);
  if (st != AGNN_OK) return st;
  if (!bytes) return fail(AGNN_EINVAL, "agnn_workspace_bytes: NULL");
  if (d->kind == AGNN_GAT) {
    *bytes = gat_workspace_bytes(*h->m.plan, gat_shape(*d));
    return AGNN_OK;
  }
  if (d->kind == AGNN_CGNN) return cg_workspace_bytes(*h->m.plan, *d, bytes);
  return av_workspace_bytes(*h->m.plan, *d, bytes);
}

agnn_status agnn_forward(agnn_model_t h, int layer, const float* W, const float* a,
                         const float* H_in, float* H_out, void* saved, void* ws, cudaStream_t s) {
  const agnn_layer_desc* d;
  agnn_status st = layer_of(h, layer, &d);
  if (st != AGNN_OK) return st;
  const Plan& p = *h->m.plan;
  if (!W || !ws || (p.n_local > 0 && (!H_in || !H_out)))
    return fail(AGNN_EINVAL, "agnn_forward: NULL W / workspace / H_in / H_out");
  if (!aligned16(W) || !aligned16(H_in) || !aligned16(H_out) || !aligned16(saved) ||
      !aligned16(ws))
    return fail(AGNN_EINVAL, "agnn_forward: pointers must be 16-byte aligned");
  if (g_profiling) prof_mark("", s);
  if (d->kind == AGNN_GAT) {
    if (!a || !aligned16(a)) return fail(AGNN_EINVAL, "agnn_forward: GAT needs an aligned `a`");
    return gat_forward(p, gat_shape(*d), W, a, H_in, H_out, saved, ws, s);
  }
  if (d->kind == AGNN_CGNN) return cg_forward(p, *d, W, H_in, H_out, saved, ws, s);
  return av_forward(p, *d, W, H_in, H_out, saved, ws, s);
}

agnn_status agnn_backward(agnn_model_t h, int layer, const float* W, const float* a,
                          const float* H_in, const void* saved, const float* dH_out, float* dH_in,
                          float* dW, float* da, void* ws, cudaStream_t s) {
  const agnn_layer_desc* d;
  agnn_status st = layer_of(h, layer, &d);
  if (st != AGNN_OK) return st;
  const Plan& p = *h->m.plan;
  if (!W || !ws || !saved || !dW || (p.n_local > 0 && (!H_in || !dH_out)))
    return fail(AGNN_EINVAL, "agnn_backward: NULL W / workspace / saved / dW / H_in / dH_out");
  if (!aligned16(W) || !aligned16(H_in) || !aligned16(dH_out) || !aligned16(dH_in) ||
      !aligned16(saved) || !aligned16(ws) || !aligned16(dW))
    return fail(AGNN_EINVAL, "agnn_backward: pointers must be 16-byte aligned");
  if (g_profiling) prof_mark("", s);
  if (d->kind == AGNN_GAT) {
    if (!a || !aligned16(a)) return fail(AGNN_EINVAL, "agnn_backward: GAT needs an aligned `a`");
    return gat_backward(p, gat_shape(*d), W, a, H_in, saved, dH_out, dH_in, dW, da, ws, s);
  }
  if (d->kind == AGNN_CGNN) return cg_backward(p, *d, W, H_in, saved, dH_out, dH_in, dW, ws, s);
  return av_backward(p, *d, W, H_in, saved, dH_out, dH_in, dW, ws, s);
}

agnn_status agnn_debug_attention(agnn_model_t h, int layer, const void* saved,
                                 const float* H_in, const int64_t* edge_pos, int64_t count,
                                 float* out, cudaStream_t s) {
  const agnn_layer_desc* d;
  agnn_status st = layer_of(h, layer, &d);
  if (st != AGNN_OK) return st;
  if (count > 0 && (!edge_pos || !out)) return fail(AGNN_EINVAL, "agnn_debug_attention: NULL");
  if (d->kind == AGNN_GAT)
    return gat_debug_alpha(*h->m.plan, gat_shape(*d), saved, edge_pos, count, out, s);
  if (d->kind == AGNN_CGNN)
    return fail(AGNN_EUNSUPPORTED, "debug_attention: a C-GNN layer has no attention");
  return av_debug_attention(*h->m.plan, *d, saved, H_in, edge_pos, count, out, s);
}

}  // extern "C"
