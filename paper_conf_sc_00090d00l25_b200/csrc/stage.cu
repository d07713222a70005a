// gllm_stage: one pipeline stage's layers on one B200 (P1) and
// the per-stage forward over one Token-Throttled mixed batch (steps a2-a12).
//
// Per forward (all on the caller's stream, nothing synchronises with the host):
//   host: validate + pack the batch metadata and the attention work lists into a pinned
//         ring slot (input prep), one H2D copy
//   prep (slot mapping O2 + RoPE table) -> [stage 0: embedding] -> per layer:
//     RMSNorm -> QKV GEMM(+bias) -> RoPE + KV append -> prefill attention | decode attention
//     -> O GEMM (+= residual) -> RMSNorm -> gate_up GEMM (SiLU*up) -> down GEMM (+= residual)
//   [last stage: final RMSNorm on sampled rows -> LM-head GEMM with argmax epilogue -> reduce]
#include <cuda_bf16.h>
#include <nccl.h>

#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "attention.cuh"
#include "common.h"
#include "gemm.cuh"
#include "kernels.cuh"
#include "kvpage.cuh"

using bf16 = __nv_bfloat16;

namespace {

#define CK(expr)                                                                                   \
  do {                                                                                             \
    cudaError_t e__ = (expr);                                                                      \
    if (e__ != cudaSuccess) return gllm::set_error(GLLM_ECUDA, "%s: %s", #expr, cudaGetErrorString(e__)); \
  } while (0)
#define RC(expr)            \
  do {                      \
    int r__ = (expr);       \
    if (r__ < 0) return r__; \
  } while (0)

constexpr uint64_t T_EMBED = 0xFFFFF0ull, T_LMHEAD = 0xFFFFF1ull;
enum Kind { K_WQ = 0, K_WK, K_WV, K_WO, K_WG, K_WU, K_WD, K_BQ, K_BK, K_BV };
inline uint64_t layer_tid(int l, int kind) { return 1 + 16 * (uint64_t)l + kind; }

// profiling categories (gllm_stage_last_timing)
enum Cat { C_TOTAL = 0, C_QKV, C_O, C_GU, C_DOWN, C_PREFILL, C_DECODE, C_ROPE, C_NORM, C_LMHEAD, C_OTHER, C_ATTN, C_N };

struct LayerW {
  bf16 *wqkv = nullptr, *wo = nullptr, *wgu = nullptr, *wd = nullptr;
  float* bqkv = nullptr;
  bf16 *kc = nullptr, *vc = nullptr;
  CUtensorMap tm_qkv, tm_o, tm_gu, tm_d;  // (the paged K / V cache needs no tensor map: kvpage.cuh)
};

constexpr int RING = 4;

// NCCL is resolved lazily with dlopen at the first communicator call, so the library never
// drags its own libnccl.so.2 into a process ahead of torch's (same soname, different version).
struct NcclApi {
  decltype(&ncclGetUniqueId) get_unique_id = nullptr;
  decltype(&ncclCommInitRank) comm_init_rank = nullptr;
  decltype(&ncclCommDestroy) comm_destroy = nullptr;
  decltype(&ncclSend) send = nullptr;
  decltype(&ncclRecv) recv = nullptr;
  decltype(&ncclGetErrorString) error_string = nullptr;
  decltype(&ncclCommCount) comm_count = nullptr;
  decltype(&ncclCommUserRank) user_rank = nullptr;
  bool ok = false;
};
NcclApi& nccl() {
  static NcclApi api = [] {
    NcclApi a;
    void* h = nullptr;
    if (const char* p = std::getenv("GLLM_NCCL_PATH")) h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);  // torch's, if loaded
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return a;
    a.get_unique_id = reinterpret_cast<decltype(a.get_unique_id)>(dlsym(h, "ncclGetUniqueId"));
    a.comm_init_rank = reinterpret_cast<decltype(a.comm_init_rank)>(dlsym(h, "ncclCommInitRank"));
    a.comm_destroy = reinterpret_cast<decltype(a.comm_destroy)>(dlsym(h, "ncclCommDestroy"));
    a.send = reinterpret_cast<decltype(a.send)>(dlsym(h, "ncclSend"));
    a.recv = reinterpret_cast<decltype(a.recv)>(dlsym(h, "ncclRecv"));
    a.error_string = reinterpret_cast<decltype(a.error_string)>(dlsym(h, "ncclGetErrorString"));
    a.comm_count = reinterpret_cast<decltype(a.comm_count)>(dlsym(h, "ncclCommCount"));
    a.user_rank = reinterpret_cast<decltype(a.user_rank)>(dlsym(h, "ncclCommUserRank"));
    a.ok = a.get_unique_id && a.comm_init_rank && a.comm_destroy && a.send && a.recv && a.error_string &&
           a.comm_count && a.user_rank;
    return a;
  }();
  return api;
}

size_t align16(size_t x) { return (x + 15) & ~size_t(15); }

// One batch's metadata, packed on the host (pinned) and copied to the device once: token ids,
// positions, cu_q, kv_len, block table, sample rows and the attention work lists.
struct Prepared {
  bool in_use = false;
  int T = 0, S = 0, NP = 0, maxblk = 0, ns = 0, n_pi = 0, n_di = 0, n_mi = 0, split_len = 16, nparts = 0;
  size_t o_ids = 0, o_pos = 0, o_cu = 0, o_kvl = 0, o_bt = 0, o_samp = 0, o_pi = 0, o_di = 0, o_mi = 0, bytes = 0;
  uint8_t* host = nullptr;
  uint8_t* dev = nullptr;
  size_t cap = 0;
  cudaEvent_t copied = nullptr;  // H2D of this slot done
  cudaEvent_t used = nullptr;    // last forward reading this slot done
};

}  // namespace

struct gllm_stage {
  gllm_model_cfg cfg{};
  int lb = 0, le = 0, kv_blocks = 0, bs = 16, max_tokens = 0, max_seqs = 0, device = 0, num_sms = 148;
  int rows_alloc = 0, seqs_alloc = 0;
  std::vector<LayerW> layers;
  bf16* embed = nullptr;
  bf16* lm_head = nullptr;
  float* final_norm = nullptr;
  CUtensorMap tm_lm;
  float* xbuf = nullptr;
  bf16 *y = nullptr, *qkv = nullptr, *attn = nullptr, *act = nullptr, *ys = nullptr;
  CUtensorMap tm_y, tm_attn, tm_act, tm_ys;
  CUtensorMap tm_yres;         // y as the residual epilogue's bf16(x) output (128 x 32 box)
  CUtensorMap tm_x;            // the residual x of the current forward (fp32, 128 x 32 box)
  const float* tm_x_base = nullptr;
  int tm_x_rows = 0;
  float2* rope_cs = nullptr;
  int32_t* slots = nullptr;
  int32_t* sampled_tmp = nullptr;
  float* gemm_ws = nullptr;  // stream-K fp32 workspace for non-additive epilogues (small T), kept zero
  float *ss_a = nullptr, *ss_b = nullptr;  // fused-RMSNorm row statistics (sum of squares of x)
  int* dec_ctr = nullptr;                  // persistent decode kernel: work counter + done counter
  float* part_val = nullptr;
  int32_t* part_idx = nullptr;
  float *part_o = nullptr, *part_ml = nullptr;
  int* part_ctr = nullptr;
  int parts_cap = 0;
  std::vector<Prepared> prep;  // [0, RING): internal ring of stage_forward; others: gllm_stage_prepare handles
  int ring_i = 0;
  std::vector<void*> allocs;
  ncclComm_t comm = nullptr;
  cudaStream_t side = nullptr;  // prefill attention runs here, concurrent with decode attention
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  int last_T = 0, last_launches = 0;
  bool profiling = false;
  bool deterministic = false;  // gllm_stage_set_deterministic: GEMM schedules with a fixed reduction order
  bool prof_serial_attn = false;  // gllm_stage_set_profiling(st, 2): attribution pass, attention in series
  // fused peer hand-off (a12, gllm_peer_*): receive ring owned here / the next stage's ring mapped here
  float* ring = nullptr;
  uint32_t* ring_flags = nullptr;
  int ring_depth = 0;
  void* peer_base = nullptr;  // IPC mapping of the next stage's ring
  float* peer_ring = nullptr;
  uint32_t* peer_flags = nullptr;
  int peer_depth = 0;
  size_t peer_slot_elems = 0;
  // slot credits (consumer -> producer): the sender owns credit[depth] (exported), the receiver maps
  // it and releases credit[tick % depth] = tick + 1 once its stage-entry kernel has read the slot
  uint32_t* credit = nullptr;       // sender: local credit flags
  void* credit_peer_base = nullptr; // receiver: IPC mapping of the previous stage's credit flags
  uint32_t* credit_peer = nullptr;
  int credit_depth = 0;
  unsigned* release_ctr = nullptr;  // receiver: CTA arrival counter of the releasing kernel (kept zero)
  const void* pending_slot = nullptr;  // receiver: slot armed by gllm_peer_ring_recv for the next forward
  uint32_t* pending_flag = nullptr;
  uint32_t pending_value = 0;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> prof_ev;
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_used = 0;
  float last_timing[C_N] = {};
  bool timing_pending = false;

  bool is_first() const { return lb == 0; }
  bool is_last() const { return le == cfg.n_layers; }
  int qd() const { return cfg.n_heads * cfg.head_dim; }
  int kd() const { return cfg.n_kv_heads * cfg.head_dim; }

  template <class T>
  int dalloc(T** p, size_t n) {
    void* q = nullptr;
    cudaError_t e = cudaMalloc(&q, std::max<size_t>(n, 1) * sizeof(T));
    if (e != cudaSuccess) {
      cudaGetLastError();
      return gllm::set_error(GLLM_ENOMEM, "cudaMalloc(%zu bytes): %s", n * sizeof(T), cudaGetErrorString(e));
    }
    allocs.push_back(q);
    *p = static_cast<T*>(q);
    return GLLM_OK;
  }
  cudaEvent_t next_ev() {
    if (ev_used == ev_pool.size()) {
      cudaEvent_t e;
      cudaEventCreate(&e);
      ev_pool.push_back(e);
    }
    return ev_pool[ev_used++];
  }
};

namespace {

struct Prof {
  gllm_stage* st;
  cudaStream_t s;
  int cat;
  cudaEvent_t a{};
  Prof(gllm_stage* st_, cudaStream_t s_, int cat_) : st(st_), s(s_), cat(cat_) {
    if (st->profiling) {
      a = st->next_ev();
      cudaEventRecord(a, s);
    }
  }
  bool closed = false;
  void close() {
    if (closed) return;
    closed = true;
    if (st->profiling) {
      cudaEvent_t b = st->next_ev();
      cudaEventRecord(b, s);
      st->prof_ev.push_back({cat, {a, b}});
    }
    if (g_sync_debug) {  // GLLM_SYNC_DEBUG=1: synchronise and log every launch group (hang triage)
      const cudaError_t e = cudaStreamSynchronize(s);
      std::fprintf(stderr, "[gllm] cat %d done: %s\n", cat, cudaGetErrorString(e));
    }
  }
  ~Prof() { close(); }
  static bool g_sync_debug;
};
bool Prof::g_sync_debug = std::getenv("GLLM_SYNC_DEBUG") != nullptr;

int gemm(gllm_stage* st, const CUtensorMap& a, const CUtensorMap& b, gllm::GemmEpi epi, int M, int N, int K,
         void* out, int ldo, const float* bias, cudaStream_t s) {
  gllm::GemmArgs g{};
  g.b_static = 1;
  g.b_tiled = 1;
  g.M = M;
  g.N = N;
  g.K = K;
  g.out = out;
  g.ldo = ldo;
  g.bias = bias;
  g.part_val = st->part_val;
  g.part_idx = st->part_idx;
  g.ws = st->gemm_ws;
  g.deterministic = st->deterministic;
  st->last_launches += 1;
  return gllm::launch_gemm(a, b, epi, g, s, st->num_sms);
}

int check_model(const gllm_model_cfg* c) {
  if (!c) return gllm::set_error(GLLM_EINVAL, "null model cfg");
  if (c->n_layers < 1 || c->hidden < 256 || c->n_heads < 1 || c->n_kv_heads < 1 || c->vocab < 256)
    return gllm::set_error(GLLM_EINVAL, "model cfg: bad sizes");
  if (c->head_dim != 64 && c->head_dim != 128) return gllm::set_error(GLLM_EINVAL, "head_dim must be 64 or 128");
  if (c->n_heads % c->n_kv_heads) return gllm::set_error(GLLM_EINVAL, "n_heads %% n_kv_heads != 0");
  const int g = c->n_heads / c->n_kv_heads;
  if (g != 1 && g != 2 && g != 4 && g != 5 && g != 8) return gllm::set_error(GLLM_EINVAL, "GQA group %d unsupported", g);
  if (c->hidden % 256) return gllm::set_error(GLLM_EINVAL, "hidden %% 256 != 0");
  if (c->intermediate % 128) return gllm::set_error(GLLM_EINVAL, "intermediate %% 128 != 0");
  if ((c->n_heads * c->head_dim) % 64 || ((c->n_heads + 2 * c->n_kv_heads) * c->head_dim) % 32)
    return gllm::set_error(GLLM_EINVAL, "q/kv dims must be multiples of 64");
  if (!(c->rms_eps > 0) || !(c->rope_theta > 1)) return gllm::set_error(GLLM_EINVAL, "bad eps/theta");
  return GLLM_OK;
}

void destroy(gllm_stage* st) {
  if (!st) return;
  cudaSetDevice(st->device);
  cudaDeviceSynchronize();
  for (void* p : st->allocs) cudaFree(p);
  for (void* p : {(void*)st->part_o, (void*)st->part_ml, (void*)st->part_ctr})
    if (p) cudaFree(p);
  for (auto& p : st->prep) {
    if (p.host) cudaFreeHost(p.host);
    if (p.dev) cudaFree(p.dev);
    if (p.copied) cudaEventDestroy(p.copied);
    if (p.used) cudaEventDestroy(p.used);
  }
  for (auto e : st->ev_pool) cudaEventDestroy(e);
  if (st->comm && nccl().ok) nccl().comm_destroy(st->comm);
  if (st->side) cudaStreamDestroy(st->side);
  if (st->ev_fork) cudaEventDestroy(st->ev_fork);
  if (st->ev_join) cudaEventDestroy(st->ev_join);
  if (st->peer_base) cudaIpcCloseMemHandle(st->peer_base);
  if (st->credit_peer_base) cudaIpcCloseMemHandle(st->credit_peer_base);
  cudaGetLastError();
  delete st;
}

int new_slot(gllm_stage* st) {
  Prepared p;
  CK(cudaEventCreateWithFlags(&p.copied, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&p.used, cudaEventDisableTiming));
  st->prep.push_back(p);
  return GLLM_OK;
}

int ensure_slot_cap(Prepared& p, size_t bytes) {
  if (bytes <= p.cap) return GLLM_OK;
  CK(cudaEventSynchronize(p.copied));
  CK(cudaEventSynchronize(p.used));
  if (p.host) cudaFreeHost(p.host);
  if (p.dev) cudaFree(p.dev);
  p.host = nullptr;
  p.dev = nullptr;
  const size_t cap = std::max<size_t>(bytes * 3 / 2, 256 << 10);
  CK(cudaMallocHost(&p.host, cap));
  CK(cudaMalloc(&p.dev, cap));
  p.cap = cap;
  return GLLM_OK;
}

int ensure_parts(gllm_stage* st, int parts) {
  if (parts <= st->parts_cap) return GLLM_OK;
  CK(cudaDeviceSynchronize());
  const int cap = std::max(parts * 2, 1024);
  const size_t G = st->cfg.n_heads / st->cfg.n_kv_heads;
  float *po = nullptr, *pm = nullptr;
  int* pc = nullptr;
  CK(cudaMalloc(&po, (size_t)cap * st->cfg.n_kv_heads * G * st->cfg.head_dim * sizeof(float)));
  CK(cudaMalloc(&pm, (size_t)cap * st->cfg.n_kv_heads * G * 2 * sizeof(float)));
  CK(cudaMalloc(&pc, (size_t)cap * st->cfg.n_kv_heads * sizeof(int)));
  CK(cudaMemset(pc, 0, (size_t)cap * st->cfg.n_kv_heads * sizeof(int)));
  if (st->part_o) cudaFree(st->part_o);
  if (st->part_ml) cudaFree(st->part_ml);
  if (st->part_ctr) cudaFree(st->part_ctr);
  st->part_o = po;
  st->part_ml = pm;
  st->part_ctr = pc;
  st->parts_cap = cap;
  return GLLM_OK;
}

}  // namespace

extern "C" {

int gllm_init_stage(const gllm_model_cfg* cfg, int32_t layer_begin, int32_t layer_end, int32_t kv_blocks,
                    int32_t block_size, int32_t max_tokens, int32_t max_seqs, int32_t device, gllm_stage** out) {
  GLLM_TRY_BEGIN
  RC(check_model(cfg));
  if (!out) return gllm::set_error(GLLM_EINVAL, "null out");
  if (layer_begin < 0 || layer_end > cfg->n_layers || layer_begin >= layer_end)
    return gllm::set_error(GLLM_EINVAL, "bad layer range [%d, %d)", layer_begin, layer_end);
  if (block_size != 16) return gllm::set_error(GLLM_EINVAL, "block_size must be 16");
  if (kv_blocks < 1 || max_tokens < 1 || max_seqs < 1 || max_seqs > max_tokens)
    return gllm::set_error(GLLM_EINVAL, "bad kv_blocks/max_tokens/max_seqs");
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
    cudaGetLastError();
    return gllm::set_error(GLLM_ECUDA, "no CUDA device %d", device);
  }
  CK(cudaSetDevice(device));
  auto* st = new gllm_stage();
  st->cfg = *cfg;
  st->lb = layer_begin;
  st->le = layer_end;
  st->kv_blocks = kv_blocks;
  st->bs = block_size;
  st->max_tokens = max_tokens;
  st->max_seqs = max_seqs;
  st->device = device;
  st->num_sms = gllm::num_sms_of_current_device();
  st->rows_alloc = std::max(128, (max_tokens + 127) / 128 * 128);
  st->seqs_alloc = std::max(128, (max_seqs + 127) / 128 * 128);
  auto fail = [&](int rc) {
    destroy(st);
    return rc;
  };
  const int H = cfg->hidden, D = cfg->head_dim, Hkv = cfg->n_kv_heads, I = cfg->intermediate, V = cfg->vocab;
  const int qd = st->qd(), kd = st->kd(), nqkv = qd + 2 * kd;
  const uint64_t seed = cfg->weight_seed;
  const float s_h = (float)std::sqrt(3.0 / H), s_q = (float)std::sqrt(3.0 / qd), s_i = (float)std::sqrt(3.0 / I);
  const float s_bias = (float)(std::sqrt(3.0) * 0.02), s_emb = (float)std::sqrt(3.0);
  cudaStream_t s0 = 0;
  const size_t kv_elems = (size_t)kv_blocks * Hkv * block_size * D;
  int rc;
  for (int l = layer_begin; l < layer_end; ++l) {
    LayerW w;
    // projection weights in the tiled layout (gemm.cuh): rows padded to a multiple of 128 (zero)
    if ((rc = st->dalloc(&w.wqkv, gllm::weight_tiled_elems(nqkv, H))) ||
        (rc = st->dalloc(&w.wo, gllm::weight_tiled_elems(H, qd))) ||
        (rc = st->dalloc(&w.wgu, gllm::weight_tiled_elems(2 * (int64_t)I, H))) ||
        (rc = st->dalloc(&w.wd, gllm::weight_tiled_elems(H, I))) ||
        (rc = st->dalloc(&w.kc, kv_elems)) || (rc = st->dalloc(&w.vc, kv_elems)))
      return fail(rc);
    if (cfg->qkv_bias && (rc = st->dalloc(&w.bqkv, nqkv))) return fail(rc);
    CK(cudaMemsetAsync(w.wqkv, 0, gllm::weight_tiled_elems(nqkv, H) * sizeof(bf16), s0));
    CK(cudaMemsetAsync(w.wo, 0, gllm::weight_tiled_elems(H, qd) * sizeof(bf16), s0));
    CK(cudaMemsetAsync(w.wgu, 0, gllm::weight_tiled_elems(2 * (int64_t)I, H) * sizeof(bf16), s0));
    CK(cudaMemsetAsync(w.wd, 0, gllm::weight_tiled_elems(H, I) * sizeof(bf16), s0));
    gllm::launch_init_bf16(w.wqkv, qd, H, seed, layer_tid(l, K_WQ), s_h, 0, 0, s0, 1);
    gllm::launch_init_bf16(w.wqkv, kd, H, seed, layer_tid(l, K_WK), s_h, 0, qd, s0, 1);
    gllm::launch_init_bf16(w.wqkv, kd, H, seed, layer_tid(l, K_WV), s_h, 0, qd + kd, s0, 1);
    gllm::launch_init_bf16(w.wo, H, qd, seed, layer_tid(l, K_WO), s_q, 0, 0, s0, 1);
    gllm::launch_init_bf16(w.wgu, I, H, seed, layer_tid(l, K_WG), s_h, 1, 0, s0, 1);
    gllm::launch_init_bf16(w.wgu, I, H, seed, layer_tid(l, K_WU), s_h, 2, 0, s0, 1);
    gllm::launch_init_bf16(w.wd, H, I, seed, layer_tid(l, K_WD), s_i, 0, 0, s0, 1);
    // The two RMSNorm gains of the layer are folded into the columns of Wqkv and Wgu
    // (W' = W diag(g)); under O4 every gain is exactly 1, so W' = W bit for bit.
    if (w.bqkv) {
      gllm::launch_init_f32(w.bqkv, qd, seed, layer_tid(l, K_BQ), s_bias, s0);
      gllm::launch_init_f32(w.bqkv + qd, kd, seed, layer_tid(l, K_BK), s_bias, s0);
      gllm::launch_init_f32(w.bqkv + qd + kd, kd, seed, layer_tid(l, K_BV), s_bias, s0);
    }
    CK(cudaMemsetAsync(w.kc, 0, kv_elems * sizeof(bf16), s0));
    CK(cudaMemsetAsync(w.vc, 0, kv_elems * sizeof(bf16), s0));
    if ((rc = gllm::make_tmap_weight_tiled(&w.tm_qkv, w.wqkv, nqkv, H)) ||
        (rc = gllm::make_tmap_weight_tiled(&w.tm_o, w.wo, H, qd)) ||
        (rc = gllm::make_tmap_weight_tiled(&w.tm_gu, w.wgu, 2 * (size_t)I, H)) ||
        (rc = gllm::make_tmap_weight_tiled(&w.tm_d, w.wd, H, I)))
      return fail(rc);
    st->layers.push_back(w);
  }
  if (st->is_first()) {
    if ((rc = st->dalloc(&st->embed, (size_t)V * H))) return fail(rc);
    gllm::launch_init_bf16(st->embed, V, H, seed, T_EMBED, s_emb, 0, 0, s0);
  }
  if (st->is_last()) {
    if ((rc = st->dalloc(&st->lm_head, gllm::weight_tiled_elems(V, H))) || (rc = st->dalloc(&st->final_norm, H)))
      return fail(rc);
    CK(cudaMemsetAsync(st->lm_head, 0, gllm::weight_tiled_elems(V, H) * sizeof(bf16), s0));
    gllm::launch_init_bf16(st->lm_head, V, H, seed, T_LMHEAD, s_h, 0, 0, s0, 1);
    gllm::launch_fill_f32(st->final_norm, H, 1.0f, s0);
    if ((rc = gllm::make_tmap_weight_tiled(&st->tm_lm, st->lm_head, V, H))) return fail(rc);
    const int ntn = (V + gllm::GEMM_BN - 1) / gllm::GEMM_BN;
    if ((rc = st->dalloc(&st->ys, (size_t)st->seqs_alloc * H)) ||
        (rc = st->dalloc(&st->part_val, (size_t)st->seqs_alloc * ntn)) ||
        (rc = st->dalloc(&st->part_idx, (size_t)st->seqs_alloc * ntn)) ||
        (rc = st->dalloc(&st->sampled_tmp, st->seqs_alloc)))
      return fail(rc);
    if ((rc = gllm::make_tmap_bf16(&st->tm_ys, st->ys, st->seqs_alloc, H, gllm::GEMM_BM))) return fail(rc);
  }
  const size_t R = st->rows_alloc;
  if ((rc = st->dalloc(&st->xbuf, R * H)) || (rc = st->dalloc(&st->y, R * H)) ||
      (rc = st->dalloc(&st->qkv, R * nqkv)) || (rc = st->dalloc(&st->attn, R * qd)) ||
      (rc = st->dalloc(&st->act, R * I)) || (rc = st->dalloc(&st->rope_cs, R * (D / 2))) ||
      (rc = st->dalloc(&st->slots, R)) ||
      // stream-K workspace for non-additive epilogues (used only for outputs <= GEMM_WS_ELEMS)
      (rc = st->dalloc(&st->gemm_ws, gllm::GEMM_WS_ELEMS)) || (rc = st->dalloc(&st->ss_a, R)) ||
      (rc = st->dalloc(&st->ss_b, R)) || (rc = st->dalloc(&st->dec_ctr, 2)) || (rc = st->dalloc(&st->release_ctr, 1)))
    return fail(rc);
  CK(cudaMemsetAsync(st->gemm_ws, 0, gllm::GEMM_WS_ELEMS * sizeof(float), s0));
  CK(cudaMemsetAsync(st->dec_ctr, 0, 2 * sizeof(int), s0));
  CK(cudaMemsetAsync(st->release_ctr, 0, sizeof(unsigned), s0));
  CK(cudaMemsetAsync(st->y, 0, R * H * sizeof(bf16), s0));
  if (!gllm::decode_tma_supported(D, cfg->n_heads / Hkv))
    return fail(gllm::set_error(GLLM_EINVAL, "decode attention: head_dim %d / GQA group %d unsupported", D,
                                cfg->n_heads / Hkv));
  CK(cudaMemsetAsync(st->attn, 0, R * qd * sizeof(bf16), s0));
  CK(cudaMemsetAsync(st->act, 0, R * I * sizeof(bf16), s0));
  if ((rc = gllm::make_tmap_bf16(&st->tm_y, st->y, R, H, gllm::GEMM_BM)) ||
      (rc = gllm::make_tmap_bf16(&st->tm_attn, st->attn, R, qd, gllm::GEMM_BM)) ||
      (rc = gllm::make_tmap_bf16(&st->tm_act, st->act, R, I, gllm::GEMM_BM)) ||
      (rc = gllm::make_tmap_res_bf16(&st->tm_yres, st->y, R, H)))
    return fail(rc);
  for (int i = 0; i < RING; ++i)
    if ((rc = new_slot(st)) < 0) return fail(rc);
  if (cudaStreamCreateWithFlags(&st->side, cudaStreamNonBlocking) != cudaSuccess ||
      cudaEventCreateWithFlags(&st->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&st->ev_join, cudaEventDisableTiming) != cudaSuccess)
    return fail(gllm::set_error(GLLM_ECUDA, "side stream / events"));
  if ((rc = ensure_parts(st, 1024)) < 0) return fail(rc);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) return fail(gllm::set_error(GLLM_ECUDA, "init: %s", cudaGetErrorString(e)));
  *out = st;
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_free_stage(gllm_stage* st) {
  destroy(st);
  return GLLM_OK;
}

}  // extern "C"

namespace {

// Validates the batch, builds the attention work lists and copies everything to the device
// slot on `s` (the early-metadata phase of the paper's dual-phase transmission, L204).
int prepare_impl(gllm_stage* st, const gllm_batch_desc* d, cudaStream_t s, Prepared& P) {
  if (!st || !d) return gllm::set_error(GLLM_EINVAL, "null argument");
  const gllm_model_cfg& c = st->cfg;
  const int T = d->num_tokens, S = d->num_seqs, NP = d->num_prefill_seqs, maxblk = d->max_blocks_per_seq;
  const int ns = d->num_samples;
  const int bs = st->bs;
  // ---------------- validation (EINVAL, never UB)
  if (T < 0 || T > st->max_tokens) return gllm::set_error(GLLM_EINVAL, "num_tokens %d > max_tokens %d", T, st->max_tokens);
  if (S < 0 || S > st->max_seqs) return gllm::set_error(GLLM_EINVAL, "num_seqs %d > max_seqs %d", S, st->max_seqs);
  if (NP < 0 || NP > S || ns < 0 || ns > S || maxblk < 0) return gllm::set_error(GLLM_EINVAL, "bad batch counts");
  P.T = T;
  P.S = S;
  P.NP = NP;
  P.maxblk = maxblk;
  P.ns = ns;
  if (T == 0) return GLLM_OK;
  if (!d->token_ids || !d->positions || !d->cu_q || !d->kv_len || !d->block_table || (ns && !d->sample_token_idx))
    return gllm::set_error(GLLM_EINVAL, "null batch array");
  if (d->cu_q[0] != 0 || d->cu_q[S] != T) return gllm::set_error(GLLM_EINVAL, "cu_q must span [0, num_tokens]");
  const int G = c.n_heads / c.n_kv_heads;
  int64_t total_pages = 0;
  for (int i = 0; i < S; ++i) {
    const int q0 = d->cu_q[i], q1 = d->cu_q[i + 1], L = d->kv_len[i], n = q1 - q0;
    if (n < 1 || (i >= NP && n != 1)) return gllm::set_error(GLLM_EINVAL, "seq %d: bad token count %d", i, n);
    if (L < n || (int64_t)(L + bs - 1) / bs > maxblk) return gllm::set_error(GLLM_EINVAL, "seq %d: bad kv_len %d", i, L);
    for (int j = 0; j < n; ++j)
      if (d->positions[q0 + j] != L - n + j) return gllm::set_error(GLLM_EINVAL, "seq %d: positions must be kv_len-n..kv_len-1", i);
    const int nb = (L + bs - 1) / bs;
    for (int j = 0; j < nb; ++j) {
      const int b = d->block_table[(size_t)i * maxblk + j];
      if (b < 0 || b >= st->kv_blocks) return gllm::set_error(GLLM_EINVAL, "seq %d: block id %d out of range", i, b);
    }
    if (i >= NP) total_pages += nb;
  }
  for (int t = 0; t < T; ++t)
    if (d->token_ids[t] < 0 || d->token_ids[t] >= c.vocab) return gllm::set_error(GLLM_EINVAL, "token id out of range");
  for (int k = 0; k < ns; ++k)
    if (d->sample_token_idx[k] < 0 || d->sample_token_idx[k] >= T) return gllm::set_error(GLLM_EINVAL, "bad sample idx");
  // ---------------- attention work lists (host, O(S))
  std::vector<gllm::PrefillItem> pitems;
  std::vector<std::pair<int, int>> pcost;  // (key tiles, item index): longest CTAs first (causal tail)
  for (int i = 0; i < NP; ++i) {
    const int n = d->cu_q[i + 1] - d->cu_q[i];
    const int rows = n * G, s0 = d->kv_len[i] - n;
    const int rpi = gllm::prefill_ws_rows_per_item();
    for (int r0 = 0; r0 < rows; r0 += rpi) {
      const int last = std::min(r0 + rpi - 1, rows - 1) / G;
      pcost.push_back({(s0 + last + 64) / 64, (int)pitems.size()});
      pitems.push_back({i, r0});
    }
  }
  std::stable_sort(pcost.begin(), pcost.end(), [](const auto& a, const auto& b) { return a.first > b.first; });
  {
    std::vector<gllm::PrefillItem> sorted(pitems.size());
    for (size_t j = 0; j < pcost.size(); ++j) sorted[j] = pitems[pcost[j].second];
    pitems.swap(sorted);
  }
  const int ND = S - NP;
  int split_pages = 1 << 30;
  if (ND > 0) {
    // Split rows longer than one warp worker's fair share of the (page, kv head) units, so the
    // persistent decode kernel's warps (8 per SM) get equal work; a split is at least 16 pages (and
    // a row at most 32 splits) so the in-place merge stays a few % of the row's bytes.  Measured on
    // B200 (profiles/r02/decode_split_ab.txt) against equal-length splits filling the workers in
    // k >= 2 rounds: the fair-share split is faster on C1 (800 rows) and on C3's few long rows.
    const int64_t W = gllm::decode_workers(st->num_sms);
    int max_pages = 1;
    for (int i = NP; i < S; ++i) max_pages = std::max(max_pages, (d->kv_len[i] + bs - 1) / bs);
    const int64_t per = (total_pages * c.n_kv_heads + W - 1) / W;
    split_pages = (int)std::min<int64_t>(256, std::max<int64_t>({16, per, (max_pages + 31) / 32}));
  }
  std::vector<gllm::DecodeItem> ditems;
  std::vector<gllm::MergeItem> merges;
  int nparts = 0;
  for (int i = NP; i < S; ++i) {
    const int nb = (d->kv_len[i] + bs - 1) / bs;
    const int nsplit = (nb + split_pages - 1) / split_pages;
    if (nsplit == 1) {
      ditems.push_back({i, 0, -1, 1});
    } else {
      merges.push_back({i, nparts, nsplit, 0});
      for (int k = 0; k < nsplit; ++k) ditems.push_back({i, k, nparts + k, nsplit});
      nparts += nsplit;
    }
  }
  // longest work items first, so the long-context CTAs do not form the tail of the grid
  std::stable_sort(ditems.begin(), ditems.end(), [&](const gllm::DecodeItem& a, const gllm::DecodeItem& b) {
    auto len = [&](const gllm::DecodeItem& it) {
      return std::min(d->kv_len[it.seq] - it.split * split_pages * bs, split_pages * bs);
    };
    return len(a) > len(b);
  });
  // ---------------- pack into the slot's pinned buffer; one H2D copy (K9)
  size_t off = 0;
  auto sect = [&](size_t bytes) {
    size_t o = off;
    off = align16(off + bytes);
    return o;
  };
  P.o_ids = sect(T * 4);
  P.o_pos = sect(T * 4);
  P.o_cu = sect((S + 1) * 4);
  P.o_kvl = sect(S * 4);
  P.o_bt = sect((size_t)S * maxblk * 4);
  P.o_samp = sect(ns * 4);
  P.o_pi = sect(pitems.size() * sizeof(gllm::PrefillItem));
  P.o_di = sect(ditems.size() * sizeof(gllm::DecodeItem));
  P.o_mi = sect(merges.size() * sizeof(gllm::MergeItem));
  P.bytes = off;
  P.n_pi = (int)pitems.size();
  P.n_di = (int)ditems.size();
  P.n_mi = (int)merges.size();
  P.split_len = split_pages * bs;
  P.nparts = nparts;
  CK(cudaSetDevice(st->device));
  RC(ensure_slot_cap(P, off));
  CK(cudaEventSynchronize(P.copied));      // the previous H2D out of this pinned buffer is done
  CK(cudaStreamWaitEvent(s, P.used, 0));   // and no queued forward still reads the device copy
  uint8_t* h = P.host;
  std::memcpy(h + P.o_ids, d->token_ids, T * 4);
  std::memcpy(h + P.o_pos, d->positions, T * 4);
  std::memcpy(h + P.o_cu, d->cu_q, (S + 1) * 4);
  std::memcpy(h + P.o_kvl, d->kv_len, S * 4);
  std::memcpy(h + P.o_bt, d->block_table, (size_t)S * maxblk * 4);
  if (ns) std::memcpy(h + P.o_samp, d->sample_token_idx, ns * 4);
  if (!pitems.empty()) std::memcpy(h + P.o_pi, pitems.data(), pitems.size() * sizeof(gllm::PrefillItem));
  if (!ditems.empty()) std::memcpy(h + P.o_di, ditems.data(), ditems.size() * sizeof(gllm::DecodeItem));
  if (!merges.empty()) std::memcpy(h + P.o_mi, merges.data(), merges.size() * sizeof(gllm::MergeItem));
  CK(cudaMemcpyAsync(P.dev, h, off, cudaMemcpyHostToDevice, s));
  CK(cudaEventRecord(P.copied, s));
  return GLLM_OK;
}

// Enqueues the stage forward of a prepared batch on `s`.
int forward_impl(gllm_stage* st, Prepared& P, const void* hidden_in, void* hidden_out, int32_t* sampled_out,
                 cudaStream_t s, float* peer_out = nullptr) {
  const gllm_model_cfg& c = st->cfg;
  const int T = P.T, S = P.S, maxblk = P.maxblk, ns = P.ns, bs = st->bs;
  st->last_launches = 0;
  st->last_T = T;
  if (T == 0) return GLLM_OK;
  if (!st->is_first() && !hidden_in) return gllm::set_error(GLLM_EINVAL, "hidden_in required on stage > 0");
  if (!st->is_last() && !hidden_out && !peer_out)
    return gllm::set_error(GLLM_EINVAL, "hidden_out required before the last stage");
  CK(cudaSetDevice(st->device));  // before ensure_parts: its buffers belong to the stage's device
  RC(ensure_parts(st, P.nparts));
  CK(cudaStreamWaitEvent(s, P.copied, 0));
  Prof p_total(st, s, C_TOTAL);
  uint8_t* m = P.dev;
  const int32_t* d_ids = reinterpret_cast<const int32_t*>(m + P.o_ids);
  const int32_t* d_pos = reinterpret_cast<const int32_t*>(m + P.o_pos);
  const int32_t* d_cu = reinterpret_cast<const int32_t*>(m + P.o_cu);
  const int32_t* d_kvl = reinterpret_cast<const int32_t*>(m + P.o_kvl);
  const int32_t* d_bt = reinterpret_cast<const int32_t*>(m + P.o_bt);
  const int32_t* d_samp = reinterpret_cast<const int32_t*>(m + P.o_samp);
  const auto* d_pi = reinterpret_cast<const gllm::PrefillItem*>(m + P.o_pi);
  const auto* d_di = reinterpret_cast<const gllm::DecodeItem*>(m + P.o_di);
  const auto* d_mi = reinterpret_cast<const gllm::MergeItem*>(m + P.o_mi);
  const int H = c.hidden, D = c.head_dim, qd = st->qd(), kd = st->kd(), nqkv = qd + 2 * kd, I = c.intermediate;
  {
    Prof p(st, s, C_OTHER);
    gllm::launch_prep(d_pos, d_cu, d_bt, T, S, maxblk, bs, st->slots, st->rope_cs, D, c.rope_theta, s);
    st->last_launches += 1;
  }
  float* x = hidden_out ? static_cast<float*>(hidden_out) : st->xbuf;
  if (st->is_first()) {
    Prof p(st, s, C_OTHER);
    gllm::launch_embed(st->embed, d_ids, x, T, H, s);
    st->last_launches += 1;
  }
  gllm::AttnArgs aa{};
  aa.q = st->qkv;
  aa.q_stride = nqkv;
  aa.Hq = c.n_heads;
  aa.Hkv = c.n_kv_heads;
  aa.D = D;
  aa.bs = bs;
  aa.cu_q = d_cu;
  aa.kv_len = d_kvl;
  aa.block_table = d_bt;
  aa.maxblk = maxblk;
  aa.out = st->attn;
  aa.part_o = st->part_o;
  aa.part_ml = st->part_ml;
  aa.part_ctr = st->part_ctr;
  aa.split_len = P.split_len;
  // Fused RMSNorm (a4): y holds bf16(x) and ss_a / ss_b the per-row sum of squares of x; the
  // consumer GEMMs (QKV, gate_up) scale their rows by rsqrt(ss/H + eps) in the epilogue and the
  // residual-add GEMMs (O, down) produce y and ss for the next norm.  Only the stage entry (and a
  // stream-K residual GEMM) needs the standalone statistics pass.  On stages after the first that
  // pass also moves hidden_in into the residual buffer (the hand-off copy-in, one read of the
  // input), and when hidden_in is a peer-ring slot its last CTA releases the slot's credit to the
  // sending stage.
  {
    Prof p(st, s, C_NORM);
    const float* src = st->is_first() ? x : static_cast<const float*>(hidden_in);
    uint32_t* rel = nullptr;
    if (!st->is_first() && hidden_in == st->pending_slot && st->pending_flag) rel = st->pending_flag;
    gllm::launch_rms_stats(src, src != x ? x : nullptr, st->y, st->ss_a, T, H, rel, st->pending_value,
                           st->release_ctr, s);
    st->pending_slot = nullptr;
    st->pending_flag = nullptr;
    st->last_launches += 1;
  }
  const float inv_h = 1.0f / (float)H;
  auto residual_gemm = [&](const CUtensorMap& ta, const CUtensorMap& tb, int K, float* ss_next,
                           float* out_peer) -> int {
    // ss_next was zeroed by the n-tile-0 epilogue of the preceding consumer GEMM (zero_rows)
    // partial tiles combine with reductions: no fused bf16(x) / sum of squares (rms_stats rebuilds
    // them); the deterministic mode also takes the statistics pass (the fused sum of squares adds
    // each tile's share atomically)
    const bool sk = gllm::gemm_uses_streamk(T, H, K, gllm::EPI_ADD_F32, st->num_sms, st->deterministic);
    const bool unfused = sk || st->deterministic;
    gllm::GemmArgs g{};
    g.b_static = 1;
    g.b_tiled = 1;
    g.deterministic = st->deterministic;
    g.M = T;
    g.N = H;
    g.K = K;
    g.out = x;
    g.ldo = H;
    g.xb_out = unfused ? nullptr : st->y;
    g.ss_out = unfused ? nullptr : ss_next;
    g.out_peer = sk ? nullptr : out_peer;  // whole tiles store the new residual rows to the peer too
    st->last_launches += 1;
    if (st->tm_x_base != x || st->tm_x_rows != T) {  // the residual's tensor map (hidden_out varies per call)
      RC(gllm::make_tmap_res_f32(&st->tm_x, x, T, H));
      st->tm_x_base = x;
      st->tm_x_rows = T;
    }
    RC(gllm::launch_gemm(ta, tb, gllm::EPI_ADD_F32, g, s, st->num_sms, &st->tm_x, &st->tm_yres));
    if (out_peer && sk)  // partial tiles reduce in place: copy the finished residual afterwards
      CK(cudaMemcpyAsync(out_peer, x, (size_t)T * H * sizeof(float), cudaMemcpyDeviceToDevice, s));
    if (unfused) {  // rebuild bf16(x) and the row sums of squares from x
      gllm::launch_rms_stats(x, nullptr, st->y, ss_next, T, H, nullptr, 0, nullptr, s);
      st->last_launches += 1;
    }
    return GLLM_OK;
  };
  for (size_t li = 0; li < st->layers.size(); ++li) {
    LayerW& w = st->layers[li];
    {
      // QKV projection with RoPE and the paged KV append fused into the epilogue (a5 + a6)
      Prof p(st, s, C_QKV);
      gllm::GemmArgs g{};
      g.b_static = 1;
      g.b_tiled = 1;
      g.M = T;
      g.N = nqkv;
      g.K = H;
      g.out = st->qkv;
      g.ldo = nqkv;
      g.bias = w.bqkv;
      g.rope_cs = st->rope_cs;
      g.slots = st->slots;
      g.kc = w.kc;
      g.vc = w.vc;
      g.q_dim = qd;
      g.kv_dim = kd;
      g.head_dim = D;
      g.n_kv_heads = c.n_kv_heads;
      g.block_size = bs;
      g.ws = st->gemm_ws;
      g.deterministic = st->deterministic;
      g.row_ss = st->ss_a;
      g.inv_h = inv_h;
      g.eps = c.rms_eps;
      g.zero_rows = st->ss_b;  // reset for the O GEMM's statistics
      st->last_launches += 1;
      RC(gllm::launch_gemm(st->tm_y, w.tm_qkv, gllm::EPI_QKV_ROPE, g, s, st->num_sms));
    }
    aa.kc = w.kc;
    aa.vc = w.vc;
    auto decode = [&](cudaStream_t ds) -> int {
      st->last_launches += 1;  // the persistent kernel merges split rows in place
      return gllm::launch_decode_attention_tma(aa, d_di, P.n_di, d_mi, P.n_mi, st->dec_ctr,
                                               st->num_sms, ds);
    };
    // Prefill rows (tensor/latency-bound) run on the side stream concurrently with the decode rows
    // (HBM-bound) on the main stream; they write disjoint rows of the attention output.
    const bool overlap = !st->prof_serial_attn && P.n_pi > 0 && P.n_di > 0;
    Prof p_attn(st, s, C_ATTN);  // span of the attention step (prefill || decode), on the main stream
    if (P.n_pi > 0) {
      cudaStream_t ps = overlap ? st->side : s;
      if (overlap) {
        CK(cudaEventRecord(st->ev_fork, s));
        CK(cudaStreamWaitEvent(ps, st->ev_fork, 0));
      }
      {
        Prof p(st, ps, C_PREFILL);
        RC(gllm::launch_prefill_attention_ws(aa, d_pi, P.n_pi, ps));
      }
      if (overlap) CK(cudaEventRecord(st->ev_join, ps));
      st->last_launches += 1;
    }
    if (overlap) {
      {
        Prof p(st, s, C_DECODE);  // the decode kernels alone (the join wait is outside)
        RC(decode(s));
      }
      CK(cudaStreamWaitEvent(s, st->ev_join, 0));
    } else if (P.n_di > 0) {
      Prof p(st, s, C_DECODE);
      RC(decode(s));
    }
    p_attn.close();
    {
      Prof p(st, s, C_O);
      RC(residual_gemm(st->tm_attn, w.tm_o, qd, st->ss_b, nullptr));
    }
    {
      Prof p(st, s, C_GU);
      gllm::GemmArgs g{};
      g.b_static = 1;
      g.b_tiled = 1;
      g.M = T;
      g.N = 2 * I;
      g.K = H;
      g.out = st->act;
      g.ldo = I;
      g.ws = st->gemm_ws;
      g.deterministic = st->deterministic;
      g.row_ss = st->ss_b;
      g.inv_h = inv_h;
      g.eps = c.rms_eps;
      g.zero_rows = st->ss_a;  // reset for the down GEMM's statistics
      st->last_launches += 1;
      RC(gllm::launch_gemm(st->tm_y, w.tm_gu, gllm::EPI_SILU_MUL, g, s, st->num_sms));
    }
    {
      Prof p(st, s, C_DOWN);
      RC(residual_gemm(st->tm_act, w.tm_d, I, st->ss_a, li + 1 == st->layers.size() ? peer_out : nullptr));
    }
  }
  if (st->is_last() && ns > 0) {
    Prof p(st, s, C_LMHEAD);
    gllm::launch_rmsnorm(x, st->final_norm, st->ys, d_samp, ns, H, c.rms_eps, s);
    RC(gemm(st, st->tm_ys, st->tm_lm, gllm::EPI_ARGMAX, ns, c.vocab, H, nullptr, 0, nullptr, s));
    const int ntn = (c.vocab + gllm::GEMM_BN - 1) / gllm::GEMM_BN;
    gllm::launch_argmax_reduce(st->part_val, st->part_idx, ns, ntn, sampled_out ? sampled_out : st->sampled_tmp, s);
    st->last_launches += 2;
  }
  CK(cudaEventRecord(P.used, s));
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return gllm::set_error(GLLM_ECUDA, "stage_forward launch: %s", cudaGetErrorString(e));
  return GLLM_OK;
}

}  // namespace

extern "C" {

int gllm_stage_forward(gllm_stage* st, const gllm_batch_desc* d, const void* hidden_in, void* hidden_out,
                       int32_t* sampled_out, void* stream) {
  GLLM_TRY_BEGIN
  if (!st || !d) return gllm::set_error(GLLM_EINVAL, "null argument");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  Prepared& P = st->prep[st->ring_i];
  st->ring_i = (st->ring_i + 1) % RING;
  RC(prepare_impl(st, d, s, P));
  return forward_impl(st, P, hidden_in, hidden_out, sampled_out, s);
  GLLM_TRY_END
}

int gllm_stage_prepare(gllm_stage* st, const gllm_batch_desc* d, void* stream, int32_t* handle) {
  GLLM_TRY_BEGIN
  if (!st || !d || !handle) return gllm::set_error(GLLM_EINVAL, "null argument");
  size_t i = RING;
  while (i < st->prep.size() && st->prep[i].in_use) ++i;
  if (i == st->prep.size()) RC(new_slot(st));
  Prepared& P = st->prep[i];
  RC(prepare_impl(st, d, reinterpret_cast<cudaStream_t>(stream), P));
  P.in_use = true;
  *handle = (int32_t)i;
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_stage_forward_prepared(gllm_stage* st, int32_t handle, const void* hidden_in, void* hidden_out,
                                int32_t* sampled_out, void* stream) {
  GLLM_TRY_BEGIN
  if (!st || handle < RING || handle >= (int32_t)st->prep.size() || !st->prep[handle].in_use)
    return gllm::set_error(GLLM_EINVAL, "bad prepared handle %d", handle);
  return forward_impl(st, st->prep[handle], hidden_in, hidden_out, sampled_out, reinterpret_cast<cudaStream_t>(stream));
  GLLM_TRY_END
}

int gllm_stage_release(gllm_stage* st, int32_t handle) {
  if (!st || handle < RING || handle >= (int32_t)st->prep.size())
    return gllm::set_error(GLLM_EINVAL, "bad prepared handle %d", handle);
  st->prep[handle].in_use = false;  // reuse waits on the slot's events
  return GLLM_OK;
}



int gllm_stage_sync(gllm_stage* st) {
  if (!st) return gllm::set_error(GLLM_EINVAL, "null stage");
  cudaSetDevice(st->device);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) return gllm::set_error(GLLM_ECUDA, "device: %s", cudaGetErrorString(e));
  return GLLM_OK;
}

int gllm_stage_set_deterministic(gllm_stage* st, int32_t on) {
  if (!st) return gllm::set_error(GLLM_EINVAL, "null stage");
  st->deterministic = on != 0;
  return GLLM_OK;
}

int gllm_stage_set_profiling(gllm_stage* st, int32_t on) {
  if (!st) return gllm::set_error(GLLM_EINVAL, "null stage");
  st->profiling = on != 0;
  st->prof_serial_attn = on == 2;
  return GLLM_OK;
}

int gllm_stage_last_timing(gllm_stage* st, float* out, int32_t n) {
  if (!st || !out) return gllm::set_error(GLLM_EINVAL, "null argument");
  float acc[C_N] = {};
  for (auto& pe : st->prof_ev) {
    CK(cudaEventSynchronize(pe.second.second));
    float ms = 0.f;
    CK(cudaEventElapsedTime(&ms, pe.second.first, pe.second.second));
    acc[pe.first] += ms;
  }
  for (int i = 0; i < n && i < C_N; ++i) out[i] = acc[i];
  st->prof_ev.clear();  // timings accumulate over forwards until read
  st->ev_used = 0;
  return GLLM_OK;
}

int gllm_stage_last_launches(gllm_stage* st, int32_t* out) {
  if (!st || !out) return gllm::set_error(GLLM_EINVAL, "null argument");
  *out = st->last_launches;
  return GLLM_OK;
}

// ---------------------------------------------------------------- NCCL hand-off (a12)
int gllm_get_unique_id(void* out128) {
  if (!out128) return gllm::set_error(GLLM_EINVAL, "null out");
  if (!nccl().ok) return gllm::set_error(GLLM_ENCCL, "libnccl.so.2 not found");
  ncclUniqueId id;
  ncclResult_t r = nccl().get_unique_id(&id);
  if (r != ncclSuccess) return gllm::set_error(GLLM_ENCCL, "ncclGetUniqueId: %s", nccl().error_string(r));
  std::memcpy(out128, &id, sizeof(id));
  return GLLM_OK;
}

int gllm_comm_init(gllm_stage* st, const void* uid, int32_t rank, int32_t world) {
  if (!st || !uid || rank < 0 || rank >= world) return gllm::set_error(GLLM_EINVAL, "bad comm_init arguments");
  if (!nccl().ok) return gllm::set_error(GLLM_ENCCL, "libnccl.so.2 not found");
  cudaSetDevice(st->device);
  ncclUniqueId id;
  std::memcpy(&id, uid, sizeof(id));
  ncclResult_t r = nccl().comm_init_rank(&st->comm, world, id, rank);
  if (r != ncclSuccess) return gllm::set_error(GLLM_ENCCL, "ncclCommInitRank: %s", nccl().error_string(r));
  return GLLM_OK;
}

int gllm_comm_size(gllm_stage* st, int32_t* nranks, int32_t* rank) {
  if (!st || !nranks || !rank) return gllm::set_error(GLLM_EINVAL, "null argument");
  if (!st->comm) return gllm::set_error(GLLM_ESTATE, "comm_size: no communicator");
  int n = 0, r = 0;
  ncclResult_t e = nccl().comm_count(st->comm, &n);
  if (e == ncclSuccess) e = nccl().user_rank(st->comm, &r);
  if (e != ncclSuccess) return gllm::set_error(GLLM_ENCCL, "ncclCommCount/UserRank: %s", nccl().error_string(e));
  *nranks = n;
  *rank = r;
  return GLLM_OK;
}

int gllm_send_hidden(gllm_stage* st, const void* buf, int32_t num_tokens, int32_t dst, void* stream) {
  if (!st || !st->comm || (!buf && num_tokens)) return gllm::set_error(GLLM_ESTATE, "send_hidden: no communicator");
  if (num_tokens == 0) return GLLM_OK;
  ncclResult_t r = nccl().send(buf, (size_t)num_tokens * st->cfg.hidden, ncclFloat32, dst, st->comm,
                            reinterpret_cast<cudaStream_t>(stream));
  if (r != ncclSuccess) return gllm::set_error(GLLM_ENCCL, "ncclSend: %s", nccl().error_string(r));
  return GLLM_OK;
}

int gllm_recv_hidden(gllm_stage* st, void* buf, int32_t num_tokens, int32_t src, void* stream) {
  if (!st || !st->comm || (!buf && num_tokens)) return gllm::set_error(GLLM_ESTATE, "recv_hidden: no communicator");
  if (num_tokens == 0) return GLLM_OK;
  ncclResult_t r = nccl().recv(buf, (size_t)num_tokens * st->cfg.hidden, ncclFloat32, src, st->comm,
                            reinterpret_cast<cudaStream_t>(stream));
  if (r != ncclSuccess) return gllm::set_error(GLLM_ENCCL, "ncclRecv: %s", nccl().error_string(r));
  return GLLM_OK;
}

// ---------------------------------------------------------------- introspection
int gllm_stage_read_weight(gllm_stage* st, int32_t layer, const char* name, int64_t row0, int64_t nrows, float* out) {
  GLLM_TRY_BEGIN
  if (!st || !name || !out || row0 < 0 || nrows < 0) return gllm::set_error(GLLM_EINVAL, "bad arguments");
  const gllm_model_cfg& c = st->cfg;
  const int H = c.hidden, I = c.intermediate, qd = st->qd(), kd = st->kd();
  const std::string n(name);
  cudaSetDevice(st->device);
  std::vector<bf16> row;
  auto copy_rows = [&](const bf16* base, int64_t rows, int64_t cols, auto phys) -> int {
    if (row0 + nrows > rows) return gllm::set_error(GLLM_EINVAL, "row range out of bounds");
    row.resize(cols);
    for (int64_t r = 0; r < nrows; ++r) {
      CK(cudaMemcpy(row.data(), base + (size_t)phys(row0 + r) * cols, cols * sizeof(bf16), cudaMemcpyDeviceToHost));
      for (int64_t j = 0; j < cols; ++j) out[r * cols + j] = __bfloat162float(row[j]);
    }
    return GLLM_OK;
  };
  // the projection weights and the LM head are stored tiled (gemm.cuh weight_tiled_index)
  auto copy_rows_tiled = [&](const bf16* base, int64_t rows, int64_t cols, auto phys) -> int {
    if (row0 + nrows > rows) return gllm::set_error(GLLM_EINVAL, "row range out of bounds");
    row.resize(64);
    for (int64_t r = 0; r < nrows; ++r) {
      const int64_t pr = phys(row0 + r);
      for (int64_t c0 = 0; c0 < cols; c0 += 64) {
        CK(cudaMemcpy(row.data(), base + gllm::weight_tiled_index(pr, c0, cols), 64 * sizeof(bf16),
                      cudaMemcpyDeviceToHost));
        for (int64_t j = 0; j < 64; ++j) out[r * cols + c0 + j] = __bfloat162float(row[j]);
      }
    }
    return GLLM_OK;
  };
  auto ident = [](int64_t r) { return r; };
  if (n == "embed") {
    if (!st->embed) return gllm::set_error(GLLM_EINVAL, "no embedding on this stage");
    return copy_rows(st->embed, c.vocab, H, ident);
  }
  if (n == "lm_head") {
    if (!st->lm_head) return gllm::set_error(GLLM_EINVAL, "no LM head on this stage");
    return copy_rows_tiled(st->lm_head, c.vocab, H, ident);
  }
  if (layer < st->lb || layer >= st->le) return gllm::set_error(GLLM_EINVAL, "layer %d not on this stage", layer);
  LayerW& w = st->layers[layer - st->lb];
  if (n == "wq") return copy_rows_tiled(w.wqkv, qd, H, ident);
  if (n == "wk") return copy_rows_tiled(w.wqkv, kd, H, [&](int64_t r) { return qd + r; });
  if (n == "wv") return copy_rows_tiled(w.wqkv, kd, H, [&](int64_t r) { return qd + kd + r; });
  if (n == "wo") return copy_rows_tiled(w.wo, H, qd, ident);
  if (n == "wg") return copy_rows_tiled(w.wgu, I, H, [](int64_t r) { return (r / 128) * 256 + r % 128; });
  if (n == "wu") return copy_rows_tiled(w.wgu, I, H, [](int64_t r) { return (r / 128) * 256 + 128 + r % 128; });
  if (n == "wd") return copy_rows_tiled(w.wd, H, I, ident);
  if (n == "bq" || n == "bk" || n == "bv") {
    if (!w.bqkv) return gllm::set_error(GLLM_EINVAL, "model has no qkv bias");
    const int64_t o = n == "bq" ? 0 : (n == "bk" ? qd : qd + kd), len = n == "bq" ? qd : kd;
    if (row0 != 0 || nrows != 1) return gllm::set_error(GLLM_EINVAL, "bias: read row 0 only");
    CK(cudaMemcpy(out, w.bqkv + o, len * sizeof(float), cudaMemcpyDeviceToHost));
    return GLLM_OK;
  }
  return gllm::set_error(GLLM_EINVAL, "unknown weight '%s'", name);
  GLLM_TRY_END
}

int gllm_stage_read_kv(gllm_stage* st, int32_t layer, const int32_t* slots, int32_t n, float* k_out, float* v_out) {
  GLLM_TRY_BEGIN
  if (!st || (!slots && n) || !k_out || !v_out) return gllm::set_error(GLLM_EINVAL, "bad arguments");
  if (layer < st->lb || layer >= st->le) return gllm::set_error(GLLM_EINVAL, "layer not on this stage");
  cudaSetDevice(st->device);
  LayerW& w = st->layers[layer - st->lb];
  const int Hkv = st->cfg.n_kv_heads, D = st->cfg.head_dim, bs = st->bs;
  std::vector<bf16> pk(bs * D), pv(bs * D);  // one page (SMEM-ready layout, kvpage.cuh)
  for (int i = 0; i < n; ++i) {
    const int64_t sl = slots[i];
    if (sl < 0 || sl >= (int64_t)st->kv_blocks * bs) return gllm::set_error(GLLM_EINVAL, "slot out of range");
    const int64_t blk = sl / bs, o = sl % bs;
    for (int h = 0; h < Hkv; ++h) {
      const int64_t page = blk * Hkv + h;
      CK(cudaMemcpy(pk.data(), w.kc + page * bs * D, bs * D * sizeof(bf16), cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(pv.data(), w.vc + page * bs * D, bs * D * sizeof(bf16), cudaMemcpyDeviceToHost));
      for (int j = 0; j < D; ++j) {
        const int64_t e = gllm::kv_page_elem(0, (int)o, j, D);
        k_out[((size_t)i * Hkv + h) * D + j] = __bfloat162float(pk[e]);
        v_out[((size_t)i * Hkv + h) * D + j] = __bfloat162float(pv[e]);
      }
    }
  }
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_stage_read_slots(gllm_stage* st, int32_t* out, int32_t n) {
  if (!st || !out || n < 0 || n > st->max_tokens) return gllm::set_error(GLLM_EINVAL, "bad arguments");
  cudaSetDevice(st->device);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(out, st->slots, n * sizeof(int32_t), cudaMemcpyDeviceToHost));
  return GLLM_OK;
}

int gllm_stage_fill_warm_kv(gllm_stage* st, int32_t n_seqs, const int64_t* req_ids, const int32_t* context_lens,
                            const int32_t* block_table, int32_t max_blocks) {
  GLLM_TRY_BEGIN
  if (!st || n_seqs < 0 || max_blocks < 0 || (n_seqs && (!req_ids || !context_lens || !block_table)))
    return gllm::set_error(GLLM_EINVAL, "fill_warm_kv: bad arguments");
  if (n_seqs == 0) return GLLM_OK;
  const int Hkv = st->cfg.n_kv_heads, D = st->cfg.head_dim, bs = st->bs;
  for (int i = 0; i < n_seqs; ++i) {
    const int n = context_lens[i];
    if (n < 1 || n > (1 << 17) || (n + bs - 1) / bs > max_blocks)
      return gllm::set_error(GLLM_EINVAL, "fill_warm_kv: seq %d context %d", i, n);
    if (req_ids[i] < 0 || ((uint64_t)(req_ids[i] + 1) << 17) * (uint64_t)(Hkv * D) > (1ull << 40))
      return gllm::set_error(GLLM_EINVAL, "fill_warm_kv: request id %lld out of the O4 index range", (long long)req_ids[i]);
    for (int j = 0; j < (n + bs - 1) / bs; ++j) {
      const int b = block_table[(size_t)i * max_blocks + j];
      if (b < 0 || b >= st->kv_blocks) return gllm::set_error(GLLM_EINVAL, "fill_warm_kv: block id %d", b);
    }
  }
  CK(cudaSetDevice(st->device));
  int64_t* d_req = nullptr;
  int32_t *d_ctx = nullptr, *d_bt = nullptr;
  const size_t bt_n = (size_t)n_seqs * max_blocks;
  CK(cudaMalloc(&d_req, n_seqs * sizeof(int64_t)));
  cudaError_t e = cudaMalloc(&d_ctx, n_seqs * sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMalloc(&d_bt, bt_n * sizeof(int32_t));
  if (e == cudaSuccess) e = cudaMemcpy(d_req, req_ids, n_seqs * sizeof(int64_t), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(d_ctx, context_lens, n_seqs * sizeof(int32_t), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) e = cudaMemcpy(d_bt, block_table, bt_n * sizeof(int32_t), cudaMemcpyHostToDevice);
  if (e == cudaSuccess) {
    for (int l = st->lb; l < st->le; ++l) {
      LayerW& w = st->layers[l - st->lb];
      gllm::launch_fill_warm_kv(w.kc, w.vc, d_req, d_ctx, d_bt, n_seqs, max_blocks, Hkv, D, bs, st->cfg.weight_seed,
                                0xEE0000ull + 2 * (uint64_t)l, 0);
    }
    e = cudaDeviceSynchronize();
  }
  cudaFree(d_req);
  cudaFree(d_ctx);
  cudaFree(d_bt);
  if (e != cudaSuccess) return gllm::set_error(GLLM_ECUDA, "fill_warm_kv: %s", cudaGetErrorString(e));
  return GLLM_OK;
  GLLM_TRY_END
}

}  // extern "C"

// ---------------------------------------------------------------- fused peer hand-off (a12)
namespace {
// ---- fused peer hand-off (a12): release flag written by one thread after the stage's last
// kernel (stream order: every store of the forward, local and peer, is complete), system scope
__global__ void peer_flag_kernel(uint32_t* flag, uint32_t value) {
  __threadfence_system();
  asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(flag), "r"(value) : "memory");
}

using PfnWaitValue32 = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
PfnWaitValue32 wait_value32() {
  static PfnWaitValue32 fn = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return (PfnWaitValue32) nullptr;
    return reinterpret_cast<PfnWaitValue32>(f);
  }();
  return fn;
}

struct PeerHandle {  // GLLM_PEER_HANDLE_BYTES
  cudaIpcMemHandle_t mem;
  int32_t depth, max_tokens, hidden, pad;
};
static_assert(sizeof(PeerHandle) <= GLLM_PEER_HANDLE_BYTES, "peer handle size");

}  // namespace

extern "C" {

int gllm_peer_ring_create(gllm_stage* st, int32_t depth, void* handle_out) {
  GLLM_TRY_BEGIN
  if (!st || !handle_out || depth < 1 || depth > 64) return gllm::set_error(GLLM_EINVAL, "peer ring: bad arguments");
  if (st->is_first()) return gllm::set_error(GLLM_ESTATE, "peer ring: the first stage receives no hidden states");
  if (st->ring) return gllm::set_error(GLLM_ESTATE, "peer ring already created");
  CK(cudaSetDevice(st->device));
  const size_t slot = (size_t)st->max_tokens * st->cfg.hidden;
  const size_t bytes = (size_t)depth * slot * sizeof(float) + 256;
  void* base = nullptr;
  CK(cudaMalloc(&base, bytes));  // one plain allocation: exportable with cudaIpcGetMemHandle
  CK(cudaMemset(base, 0, bytes));
  st->allocs.push_back(base);
  st->ring_flags = static_cast<uint32_t*>(base);  // [depth] flags in the first 256 B
  st->ring = reinterpret_cast<float*>(static_cast<uint8_t*>(base) + 256);
  st->ring_depth = depth;
  PeerHandle h{};
  CK(cudaIpcGetMemHandle(&h.mem, base));
  h.depth = depth;
  h.max_tokens = st->max_tokens;
  h.hidden = st->cfg.hidden;
  std::memset(handle_out, 0, GLLM_PEER_HANDLE_BYTES);
  std::memcpy(handle_out, &h, sizeof(h));
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_peer_ring_open(gllm_stage* st, const void* handle, void* credit_handle_out) {
  GLLM_TRY_BEGIN
  if (!st || !handle || !credit_handle_out) return gllm::set_error(GLLM_EINVAL, "peer ring open: null argument");
  if (st->is_last()) return gllm::set_error(GLLM_ESTATE, "peer ring open: the last stage sends no hidden states");
  if (st->peer_base) return gllm::set_error(GLLM_ESTATE, "peer ring already open");
  PeerHandle h;
  std::memcpy(&h, handle, sizeof(h));
  if (h.depth < 1 || h.hidden != st->cfg.hidden || h.max_tokens < st->max_tokens)
    return gllm::set_error(GLLM_EINVAL, "peer ring: shape mismatch (hidden %d vs %d, max_tokens %d vs %d)", h.hidden,
                           st->cfg.hidden, h.max_tokens, st->max_tokens);
  CK(cudaSetDevice(st->device));
  void* base = nullptr;
  CK(cudaIpcOpenMemHandle(&base, h.mem, cudaIpcMemLazyEnablePeerAccess));
  st->peer_base = base;
  st->peer_flags = static_cast<uint32_t*>(base);
  st->peer_ring = reinterpret_cast<float*>(static_cast<uint8_t*>(base) + 256);
  st->peer_depth = h.depth;
  st->peer_slot_elems = (size_t)h.max_tokens * h.hidden;
  // the slot credits live here (the waiter's memory, like the ready flags on the receiver's side);
  // the receiver maps them with gllm_peer_credit_open and releases each slot after reading it
  void* cb = nullptr;
  CK(cudaMalloc(&cb, 256));
  CK(cudaMemset(cb, 0, 256));
  st->allocs.push_back(cb);
  st->credit = static_cast<uint32_t*>(cb);
  PeerHandle ch{};
  CK(cudaIpcGetMemHandle(&ch.mem, cb));
  ch.depth = h.depth;
  ch.max_tokens = h.max_tokens;
  ch.hidden = h.hidden;
  std::memset(credit_handle_out, 0, GLLM_PEER_HANDLE_BYTES);
  std::memcpy(credit_handle_out, &ch, sizeof(ch));
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_stage_forward_prepared_peer(gllm_stage* st, int32_t handle, const void* hidden_in, int64_t tick,
                                     void* stream) {
  GLLM_TRY_BEGIN
  if (!st || handle < RING || handle >= (int32_t)st->prep.size() || !st->prep[handle].in_use)
    return gllm::set_error(GLLM_EINVAL, "bad prepared handle %d", handle);
  if (!st->peer_base) return gllm::set_error(GLLM_ESTATE, "peer ring not open");
  if (tick < 0) return gllm::set_error(GLLM_EINVAL, "negative tick");
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  const int slot = (int)(tick % st->peer_depth);
  if (tick >= st->peer_depth && st->prep[handle].T > 0) {
    // the slot last carried tick - depth: wait until the receiver has read it (credit >= tick - depth + 1)
    PfnWaitValue32 wv = wait_value32();
    if (!wv) return gllm::set_error(GLLM_ECUDA, "cuStreamWaitValue32 unavailable");
    CK(cudaSetDevice(st->device));
    const CUresult r = wv(reinterpret_cast<CUstream>(s), reinterpret_cast<CUdeviceptr>(st->credit + slot),
                          (cuuint32_t)(tick - st->peer_depth + 1), CU_STREAM_WAIT_VALUE_GEQ);
    if (r != CUDA_SUCCESS) return gllm::set_error(GLLM_ECUDA, "cuStreamWaitValue32 (credit) failed (%d)", (int)r);
  }
  float* dst = st->peer_ring + (size_t)slot * st->peer_slot_elems;
  RC(forward_impl(st, st->prep[handle], hidden_in, nullptr, nullptr, s, dst));
  if (st->prep[handle].T > 0) {
    peer_flag_kernel<<<1, 1, 0, s>>>(st->peer_flags + slot, (uint32_t)(tick + 1));
    st->last_launches += 1;
    CK(cudaGetLastError());
  }
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_peer_ring_recv(gllm_stage* st, int64_t tick, void* stream, void** slot_out) {
  GLLM_TRY_BEGIN
  if (!st || !slot_out || tick < 0) return gllm::set_error(GLLM_EINVAL, "peer recv: bad arguments");
  if (!st->ring) return gllm::set_error(GLLM_ESTATE, "peer ring not created");
  PfnWaitValue32 wv = wait_value32();
  if (!wv) return gllm::set_error(GLLM_ECUDA, "cuStreamWaitValue32 unavailable");
  const int slot = (int)(tick % st->ring_depth);
  CK(cudaSetDevice(st->device));
  // (int32)(flag - (tick + 1)) >= 0: the sender released this slot for tick (or a later one)
  const CUresult r = wv(reinterpret_cast<CUstream>(stream), reinterpret_cast<CUdeviceptr>(st->ring_flags + slot),
                        (cuuint32_t)(tick + 1), CU_STREAM_WAIT_VALUE_GEQ);
  if (r != CUDA_SUCCESS) return gllm::set_error(GLLM_ECUDA, "cuStreamWaitValue32 failed (%d)", (int)r);
  *slot_out = st->ring + (size_t)slot * st->max_tokens * st->cfg.hidden;
  if (st->credit_peer) {  // the next forward reading this slot releases its credit (rms_stats' last CTA)
    st->pending_slot = *slot_out;
    st->pending_flag = st->credit_peer + slot;
    st->pending_value = (uint32_t)(tick + 1);
  }
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_peer_credit_open(gllm_stage* st, const void* credit_handle) {
  GLLM_TRY_BEGIN
  if (!st || !credit_handle) return gllm::set_error(GLLM_EINVAL, "peer credit open: null argument");
  if (!st->ring) return gllm::set_error(GLLM_ESTATE, "peer credit open: create the receive ring first");
  if (st->credit_peer_base) return gllm::set_error(GLLM_ESTATE, "peer credits already open");
  PeerHandle h;
  std::memcpy(&h, credit_handle, sizeof(h));
  if (h.depth != st->ring_depth || h.hidden != st->cfg.hidden)
    return gllm::set_error(GLLM_EINVAL, "peer credit: depth %d / hidden %d do not match the ring", h.depth, h.hidden);
  CK(cudaSetDevice(st->device));
  void* base = nullptr;
  CK(cudaIpcOpenMemHandle(&base, h.mem, cudaIpcMemLazyEnablePeerAccess));
  st->credit_peer_base = base;
  st->credit_peer = static_cast<uint32_t*>(base);
  return GLLM_OK;
  GLLM_TRY_END
}

}  // extern "C"
