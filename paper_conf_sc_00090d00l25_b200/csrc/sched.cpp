// Token-Throttling scheduler + paged-KV block manager (host, C++).
//
// Implements PAPER.md §3.1 (Eq.1-3 + the L165 threshold), §3.2 (Eq.4), the
// decoupled merge of L125/L131-L143, chunked prefill + CPP (L81, L92, L212)
// and the shared page tables of L136/L198, under the canonical readings
// R1-R18 of DESIGN.md §3.  Decisions and slot mapping must equal the oracle
// (oracle/scheduler.py, an independent Python implementation) bit for bit;
// tests/test_sched_parity.py diffs the canonical traces.
#include <algorithm>
#include <cstring>
#include <functional>
#include <map>
#include <memory>
#include <queue>
#include <unordered_map>
#include <unordered_set>
#include <vector>

#include "common.h"

namespace {

struct Req {
  int64_t id = 0, arrival = 0;
  int32_t orig_len = 0, output_len = 0;
  std::vector<int32_t> ids;
  int32_t prefill_len = 0, sched_prompt = 0, done_prompt = 0, gen = 0;
  std::vector<int32_t> blocks;
  int32_t inflight = 0;
  int64_t ready_tick = 0;
  bool finished = false;
  bool decode_phase() const { return !finished && done_prompt == prefill_len; }
  bool waiting() const { return !finished && sched_prompt < prefill_len; }
};

struct Chunk { Req* r; int32_t start, len; bool completes; };
struct Decode { Req* r; int32_t pos; };

struct BatchStore {
  int64_t tick = 0;
  int32_t P = 0, D = 0;
  std::vector<Chunk> chunks;
  std::vector<Decode> decodes;
  std::vector<int32_t> token_ids, positions, slots, cu_q, kv_len, block_table, samples;
  std::vector<int64_t> seq_ids;
  int32_t maxblk = 0;
  std::vector<int32_t> sampled;
};

int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

}  // namespace

struct gllm_sched {
  gllm_sched_cfg cfg;
  int64_t tick = 0;
  std::priority_queue<int32_t, std::vector<int32_t>, std::greater<int32_t>> free_pool;
  std::vector<std::unique_ptr<Req>> storage;
  std::unordered_set<int64_t> ids_seen;
  std::vector<Req*> pending;      // not yet admitted, sorted by (arrival, id) lazily
  size_t next_arrival = 0;
  bool pending_dirty = false;
  std::vector<Req*> admitted;     // admission order
  std::map<int64_t, BatchStore> inflight;
  int64_t preemptions = 0, finished = 0, admitted_total = 0;
  std::vector<int64_t> trace;

  int32_t alloc(Req* r, std::vector<std::pair<int64_t, int32_t>>* allocs) {
    int32_t b = free_pool.top();  // lowest-numbered free block (R8)
    free_pool.pop();
    r->blocks.push_back(b);
    if (allocs) allocs->push_back({r->id, b});
    return b;
  }
  void release(Req* r) {
    for (int32_t b : r->blocks) free_pool.push(b);
    r->blocks.clear();
  }
};

namespace {

int32_t throttle_prefill(const gllm_sched_cfg& c, int64_t wp, int64_t free_blocks) {
  const int64_t n = c.num_blocks, num = c.kvthresh_num, den = c.kvthresh_den;
  if (wp == 0 || free_blocks * den < num * n) return 0;  // KV_free < KV_thresh: suspend (L165)
  int64_t cap = ((int64_t)c.maxp * (free_blocks * den - num * n)) / (n * (den - num));
  int64_t p = std::min(wp / c.iterp, cap);               // Eq.3 inner min (WT vs UT)
  p = std::max(p, (int64_t)c.minp);                      // Eq.3 outer max (#MinP)
  return (int32_t)std::min(p, wp);                       // R11: cannot exceed #WP
}

int32_t throttle_decode(const gllm_sched_cfg& c, int64_t rd) {
  return (int32_t)ceil_div(rd, c.pp_depth);  // Eq.4 with ceil (R6)
}

int check_cfg(const gllm_sched_cfg* c) {
  if (!c) return gllm::set_error(GLLM_EINVAL, "null cfg");
  if (c->iterp < 1 || c->maxp < 0 || c->minp < 0 || c->pp_depth < 1 || c->num_blocks < 1 ||
      c->block_size < 1 || c->max_seqs < 1)
    return gllm::set_error(GLLM_EINVAL, "scheduler cfg: non-positive size");
  if (c->kvthresh_den < 1 || c->kvthresh_num < 0 || c->kvthresh_num >= c->kvthresh_den)
    return gllm::set_error(GLLM_EINVAL, "scheduler cfg: KV_thresh must be in [0,1)");
  if (c->policy != 0 && c->policy != 1) return gllm::set_error(GLLM_EINVAL, "unknown policy");
  return GLLM_OK;
}

void retire(gllm_sched* s, BatchStore& b) {
  std::vector<Req*> touched;
  for (auto& c : b.chunks) {
    Req* r = c.r;
    r->done_prompt += c.len;
    r->inflight -= 1;
    if (r->done_prompt == r->prefill_len) {  // prompt completes: first output token (R2)
      r->gen += 1;
      r->ready_tick = s->tick;
    }
    touched.push_back(r);
  }
  for (auto& d : b.decodes) {
    Req* r = d.r;
    r->gen += 1;
    r->inflight -= 1;
    r->ready_tick = s->tick;
    touched.push_back(r);
  }
  bool any = false;
  for (Req* r : touched) {
    if (!r->finished && r->gen >= r->output_len) {  // fixed output length (R3)
      r->finished = true;
      s->release(r);
      s->finished += 1;
      any = true;
    }
  }
  if (any) {
    s->admitted.erase(std::remove_if(s->admitted.begin(), s->admitted.end(),
                                     [](Req* r) { return r->finished; }),
                      s->admitted.end());
  }
}

}  // namespace

extern "C" {

int gllm_throttle_counts(const gllm_sched_cfg* cfg, int64_t wp, int64_t rd, int32_t free_blocks,
                         int32_t* P, int32_t* D) {
  int rc = check_cfg(cfg);
  if (rc) return rc;
  if (wp < 0 || rd < 0 || free_blocks < 0 || free_blocks > cfg->num_blocks)
    return gllm::set_error(GLLM_EINVAL, "throttle_counts: bad statistics");
  if (P) *P = throttle_prefill(*cfg, wp, free_blocks);
  if (D) *D = throttle_decode(*cfg, rd);
  return GLLM_OK;
}

int gllm_sched_create(const gllm_sched_cfg* cfg, gllm_sched** out) {
  GLLM_TRY_BEGIN
  int rc = check_cfg(cfg);
  if (rc) return rc;
  if (!out) return gllm::set_error(GLLM_EINVAL, "null out");
  auto* s = new gllm_sched();
  s->cfg = *cfg;
  std::vector<int32_t> all(cfg->num_blocks);
  for (int32_t i = 0; i < cfg->num_blocks; ++i) all[i] = i;
  s->free_pool = decltype(s->free_pool)(std::greater<int32_t>(), std::move(all));
  *out = s;
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_sched_free(gllm_sched* s) {
  delete s;
  return GLLM_OK;
}

int gllm_sched_add_request(gllm_sched* s, int64_t req_id, int64_t arrival_tick, int32_t prompt_len,
                           int32_t output_len, const int32_t* token_ids) {
  GLLM_TRY_BEGIN
  if (!s || !token_ids) return gllm::set_error(GLLM_EINVAL, "null argument");
  if (prompt_len < 1 || output_len < 1) return gllm::set_error(GLLM_EINVAL, "prompt/output length < 1");
  if (!s->ids_seen.insert(req_id).second) return gllm::set_error(GLLM_EINVAL, "duplicate req_id %lld", (long long)req_id);
  auto r = std::make_unique<Req>();
  r->id = req_id;
  r->arrival = arrival_tick;
  r->orig_len = prompt_len;
  r->output_len = output_len;
  r->prefill_len = prompt_len;
  r->ids.assign(token_ids, token_ids + (prompt_len + output_len - 1));
  s->pending.push_back(r.get());
  s->storage.push_back(std::move(r));
  s->pending_dirty = true;
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_sched_add_warm(gllm_sched* s, int64_t req_id, int32_t context_len, int32_t remaining_out,
                        const int32_t* token_ids) {
  GLLM_TRY_BEGIN
  if (!s || !token_ids) return gllm::set_error(GLLM_EINVAL, "null argument");
  if (context_len < 1 || remaining_out < 0) return gllm::set_error(GLLM_EINVAL, "bad warm lengths");
  if (!s->ids_seen.insert(req_id).second) return gllm::set_error(GLLM_EINVAL, "duplicate req_id");
  const int64_t need = ceil_div(context_len, s->cfg.block_size);
  if ((int64_t)s->free_pool.size() < need) return gllm::set_error(GLLM_ENOMEM, "KV pool too small for warm sequence");
  auto r = std::make_unique<Req>();
  r->id = req_id;
  r->arrival = -1;
  r->orig_len = context_len;
  r->output_len = remaining_out + 1;
  r->prefill_len = r->sched_prompt = r->done_prompt = context_len;
  r->gen = 1;
  r->ids.assign(token_ids, token_ids + (context_len + remaining_out));
  for (int64_t i = 0; i < need; ++i) s->alloc(r.get(), nullptr);
  s->admitted.push_back(r.get());
  s->admitted_total += 1;
  s->storage.push_back(std::move(r));
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_build_batch(gllm_sched* s, gllm_batch_desc* out) {
  GLLM_TRY_BEGIN
  if (!s || !out) return gllm::set_error(GLLM_EINVAL, "null argument");
  const gllm_sched_cfg& cfg = s->cfg;
  const int32_t bs = cfg.block_size;
  const int64_t k = s->tick;
  // 1. retire k - PP (R1)
  auto it = s->inflight.find(k - cfg.pp_depth);
  if (it != s->inflight.end()) {
    retire(s, it->second);
    s->inflight.erase(it);
  }
  // 2. admit arrivals (R4)
  if (s->pending_dirty) {
    std::stable_sort(s->pending.begin() + s->next_arrival, s->pending.end(), [](Req* a, Req* b) {
      return a->arrival != b->arrival ? a->arrival < b->arrival : a->id < b->id;
    });
    s->pending_dirty = false;
  }
  while (s->next_arrival < s->pending.size() && s->pending[s->next_arrival]->arrival <= k) {
    s->admitted.push_back(s->pending[s->next_arrival++]);
    s->admitted_total += 1;
  }
  // 3. statistics (R5)
  int64_t rd = 0, wp = 0;
  for (Req* r : s->admitted) {
    if (r->decode_phase()) rd += 1;
    if (r->waiting()) wp += r->prefill_len - r->sched_prompt;
  }
  const int64_t free0 = (int64_t)s->free_pool.size();
  std::vector<std::pair<int64_t, int32_t>> allocs;
  std::vector<int64_t> preempted;
  std::unordered_set<int64_t> selected;
  BatchStore b;
  b.tick = k;
  // 4. decode selection (Eq.4; R6-R9; R14)
  const int32_t d_cnt = cfg.policy == 1 ? (int32_t)rd : throttle_decode(cfg, rd);
  std::vector<Req*> ready;
  for (Req* r : s->admitted)
    if (r->decode_phase() && r->inflight == 0) ready.push_back(r);
  std::sort(ready.begin(), ready.end(), [](Req* a, Req* b) {
    if (a->ready_tick != b->ready_tick) return a->ready_tick < b->ready_tick;
    if (a->arrival != b->arrival) return a->arrival < b->arrival;
    return a->id < b->id;
  });
  const size_t n_try = std::min<size_t>((size_t)d_cnt, ready.size());
  for (size_t i = 0; i < n_try; ++i) {
    Req* r = ready[i];
    if (!r->decode_phase()) continue;  // preempted earlier this tick
    const int32_t pos = r->orig_len + r->gen - 1;
    if ((int64_t)r->blocks.size() * bs <= pos) {
      if (s->free_pool.empty()) {
        // victim: latest (arrival, id) running request, not in flight, not selected (R14)
        Req* victim = nullptr;
        for (Req* c : s->admitted) {
          if (c->blocks.empty() || c->inflight != 0 || c == r || selected.count(c->id)) continue;
          if (!victim || c->arrival > victim->arrival ||
              (c->arrival == victim->arrival && c->id > victim->id))
            victim = c;
        }
        if (!victim) continue;
        s->release(victim);
        victim->prefill_len = victim->orig_len + victim->gen;
        victim->sched_prompt = victim->done_prompt = 0;
        s->preemptions += 1;
        preempted.push_back(victim->id);
      }
      s->alloc(r, &allocs);
    }
    b.decodes.push_back({r, pos});
    selected.insert(r->id);
  }
  // 5. prefill count (Eq.3 + L165; R10-R12)
  int32_t p_cnt;
  if (cfg.policy == 1)
    p_cnt = (int32_t)std::min<int64_t>(std::max<int64_t>(cfg.token_budget - (int64_t)b.decodes.size(), 0), wp);
  else
    p_cnt = throttle_prefill(cfg, wp, free0);
  // 6. prefill selection, FCFS with CPP (R13)
  int64_t running = 0;
  std::vector<Req*> waiting;
  for (Req* r : s->admitted) {
    if (!r->blocks.empty() || r->sched_prompt > 0) running += 1;
    if (r->waiting()) waiting.push_back(r);
  }
  std::sort(waiting.begin(), waiting.end(), [](Req* a, Req* b) {
    return a->arrival != b->arrival ? a->arrival < b->arrival : a->id < b->id;
  });
  int64_t p_left = p_cnt;
  for (Req* r : waiting) {
    if (p_left == 0) break;
    const bool fresh = r->blocks.empty() && r->sched_prompt == 0;
    if (fresh && running >= cfg.max_seqs) continue;
    const int64_t remaining = r->prefill_len - r->sched_prompt;
    const int64_t want = std::min(remaining, p_left);
    const int64_t capacity = ((int64_t)r->blocks.size() + (int64_t)s->free_pool.size()) * bs - r->sched_prompt;
    const int64_t c = std::min(want, capacity);
    if (c <= 0) break;
    const int64_t need = ceil_div(r->sched_prompt + c, bs) - (int64_t)r->blocks.size();
    for (int64_t j = 0; j < need; ++j) s->alloc(r, &allocs);
    if (fresh) running += 1;
    b.chunks.push_back({r, r->sched_prompt, (int32_t)c, r->sched_prompt + c == r->prefill_len});
    r->sched_prompt += (int32_t)c;
    p_left -= c;
    if (c < want) break;
  }
  // 7. layout (R15): prefill chunks, then decodes
  b.P = p_cnt;
  b.D = d_cnt;
  b.cu_q.push_back(0);
  std::vector<const Req*> rows_req;
  std::vector<int32_t> rows_n;
  for (auto& c : b.chunks) {
    for (int32_t p = c.start; p < c.start + c.len; ++p) {
      b.token_ids.push_back(c.r->ids[p]);
      b.positions.push_back(p);
      b.slots.push_back(c.r->blocks[p / bs] * bs + p % bs);  // O2
    }
    b.cu_q.push_back(b.cu_q.back() + c.len);
    b.kv_len.push_back(c.start + c.len);
    if (c.completes) b.samples.push_back(b.cu_q.back() - 1);
    b.seq_ids.push_back(c.r->id);
    rows_req.push_back(c.r);
    rows_n.push_back((int32_t)ceil_div(c.start + c.len, bs));
    c.r->inflight += 1;
  }
  for (auto& d : b.decodes) {
    b.token_ids.push_back(d.r->ids[d.pos]);
    b.positions.push_back(d.pos);
    b.slots.push_back(d.r->blocks[d.pos / bs] * bs + d.pos % bs);
    b.cu_q.push_back(b.cu_q.back() + 1);
    b.kv_len.push_back(d.pos + 1);
    b.samples.push_back(b.cu_q.back() - 1);
    b.seq_ids.push_back(d.r->id);
    rows_req.push_back(d.r);
    rows_n.push_back((int32_t)ceil_div(d.pos + 1, bs));
    d.r->inflight += 1;
  }
  b.maxblk = 0;
  for (int32_t n : rows_n) b.maxblk = std::max(b.maxblk, n);
  b.block_table.assign(rows_req.size() * (size_t)b.maxblk, -1);
  for (size_t i = 0; i < rows_req.size(); ++i)
    for (int32_t j = 0; j < rows_n[i]; ++j) b.block_table[i * b.maxblk + j] = rows_req[i]->blocks[j];
  // canonical trace (== oracle.scheduler.trace_bytes)
  auto& t = s->trace;
  t.clear();
  const int64_t T = (int64_t)b.token_ids.size();
  t.insert(t.end(), {k, (int64_t)p_cnt, (int64_t)d_cnt, rd, wp, free0, (int64_t)s->free_pool.size(),
                     (int64_t)b.chunks.size(), (int64_t)b.decodes.size(), (int64_t)preempted.size(),
                     (int64_t)allocs.size(), T, (int64_t)b.samples.size()});
  for (auto& c : b.chunks) t.insert(t.end(), {c.r->id, (int64_t)c.start, (int64_t)c.len});
  for (auto& d : b.decodes) t.insert(t.end(), {d.r->id, (int64_t)d.pos});
  for (int64_t v : preempted) t.push_back(v);
  for (auto& a : allocs) t.insert(t.end(), {a.first, (int64_t)a.second});
  for (int32_t v : b.slots) t.push_back(v);
  for (int32_t v : b.samples) t.push_back(v);

  auto& st = s->inflight[k];
  st = std::move(b);
  s->tick += 1;
  std::memset(out, 0, sizeof(*out));
  out->tick = k;
  out->P = st.P;
  out->D = st.D;
  int32_t np = 0;
  for (auto& c : st.chunks) np += c.len;
  out->num_prefill_tokens = np;
  out->num_decode_tokens = (int32_t)st.decodes.size();
  out->num_tokens = (int32_t)st.token_ids.size();
  out->num_seqs = (int32_t)(st.chunks.size() + st.decodes.size());
  out->num_prefill_seqs = (int32_t)st.chunks.size();
  out->max_blocks_per_seq = st.maxblk;
  out->num_samples = (int32_t)st.samples.size();
  out->token_ids = st.token_ids.data();
  out->positions = st.positions.data();
  out->slot_mapping = st.slots.data();
  out->cu_q = st.cu_q.data();
  out->kv_len = st.kv_len.data();
  out->block_table = st.block_table.data();
  out->sample_token_idx = st.samples.data();
  out->seq_req_ids = st.seq_ids.data();
  return out->num_tokens == 0 ? GLLM_EMPTY : GLLM_OK;
  GLLM_TRY_END
}

int gllm_retire_batch(gllm_sched* s, int64_t tick, const int32_t* sampled_ids) {
  GLLM_TRY_BEGIN
  if (!s) return gllm::set_error(GLLM_EINVAL, "null sched");
  auto it = s->inflight.find(tick);
  if (it == s->inflight.end()) return gllm::set_error(GLLM_ESTATE, "tick %lld not in flight", (long long)tick);
  if (sampled_ids) it->second.sampled.assign(sampled_ids, sampled_ids + it->second.samples.size());
  return GLLM_OK;
  GLLM_TRY_END
}

int gllm_sched_done(const gllm_sched* s) {
  if (!s) return 0;
  return s->next_arrival >= s->pending.size() && s->admitted.empty() ? 1 : 0;
}

int gllm_sched_stats(const gllm_sched* s, int64_t* out6) {
  if (!s || !out6) return gllm::set_error(GLLM_EINVAL, "null argument");
  int64_t running = 0;
  for (Req* r : s->admitted)
    if (!r->blocks.empty()) running += 1;
  out6[0] = s->tick;
  out6[1] = running;
  out6[2] = (int64_t)s->free_pool.size();
  out6[3] = s->preemptions;
  out6[4] = s->finished;
  out6[5] = s->admitted_total;
  return GLLM_OK;
}

int gllm_sched_trace(gllm_sched* s, void* buf, size_t cap, size_t* used) {
  if (!s || !used) return gllm::set_error(GLLM_EINVAL, "null argument");
  const size_t n = s->trace.size() * sizeof(int64_t);
  *used = n;
  if (cap < n || (!buf && n)) return gllm::set_error(GLLM_EINVAL, "trace buffer too small (%zu < %zu)", cap, n);
  if (n) std::memcpy(buf, s->trace.data(), n);
  return GLLM_OK;
}

}  // extern "C"
