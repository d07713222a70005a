// Token-Throttling scheduler + paged-KV block manager (host, C++).
//
// Implements PAPER.md §3.1 (Eq.1-3 + the L165 threshold), §3.2 (Eq.4), the
// decoupled merge of L125/L131-L143, chunked prefill + CPP (L81, L92, L212)
// and the shared page tables of L136/L198, under the canonical readings
// R1-R18 of DESIGN.md §3.  Decisions and slot mapping must equal the oracle
// (oracle/scheduler.py, an independent Python implementation) bit for bit;
// tests/test_sched_parity.py diffs the canonical traces.
//
// Cost per tick is proportional to the work scheduled, not to the number of
// admitted requests: #WP, #RD and the running count are maintained
// incrementally, waiting prompts sit in an (arrival, id)-ordered queue and
// ready decodes in a (ready_tick, arrival, id)-ordered FIFO.  Under overload
// (the C1 stream at PP=1) thousands of prompts wait, which made the plain
// O(admitted) scans dominate the paper's 0.045 ms budget (L212).
#include <algorithm>
#include <cstring>
#include <deque>
#include <functional>
#include <map>
#include <memory>
#include <queue>
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
  int64_t sel_tick = -1;  // tick in which the request was selected as a decode (R14 exclusion)
  int64_t ready_tick = 0;
  bool finished = false;
  bool in_waitq = false;  // present in gllm_sched::waitq (possibly stale)
  bool decode_phase() const { return !finished && done_prompt == prefill_len; }
  bool waiting() const { return !finished && sched_prompt < prefill_len; }
};

bool by_arrival(const Req* a, const Req* b) { return a->arrival != b->arrival ? a->arrival < b->arrival : a->id < b->id; }
bool by_ready(const Req* a, const Req* b) {
  if (a->ready_tick != b->ready_tick) return a->ready_tick < b->ready_tick;
  return by_arrival(a, b);
}

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
  // for the canonical trace (built on demand by gllm_sched_trace)
  int64_t rd = 0, wp = 0, free0 = 0, free1 = 0;
  std::vector<int64_t> preempted;
  std::vector<std::pair<int64_t, int32_t>> allocs;
};

int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

}  // namespace

struct gllm_sched {
  gllm_sched_cfg cfg;
  int64_t tick = 0;
  std::priority_queue<int32_t, std::vector<int32_t>, std::greater<int32_t>> free_pool;
  std::vector<std::unique_ptr<Req>> storage;
  std::unordered_set<int64_t> ids_seen;
  std::vector<Req*> pending;  // not yet admitted, sorted by (arrival, id) lazily
  size_t next_arrival = 0;
  bool pending_dirty = false;
  std::vector<Req*> active;   // admitted, not finished (lazily compacted); victim search only
  size_t active_finished = 0;
  std::vector<Req*> waitq;    // waiting prompts in (arrival, id) order (lazily compacted)
  size_t waitq_stale = 0;
  std::deque<Req*> readyq;    // decode-phase, not in flight, (ready_tick, arrival, id) order
  int64_t wp = 0, rd = 0, running = 0;
  std::map<int64_t, BatchStore> inflight;
  std::vector<BatchStore> spare;  // retired batches, recycled so their buffers keep their capacity
  int64_t preemptions = 0, finished = 0, admitted_total = 0;
  int64_t last_tick = -1;

  int32_t alloc(Req* r, std::vector<std::pair<int64_t, int32_t>>* allocs) {
    int32_t b = free_pool.top();  // lowest-numbered free block (R8)
    free_pool.pop();
    if (r->blocks.empty()) running += 1;
    r->blocks.push_back(b);
    if (allocs) allocs->push_back({r->id, b});
    return b;
  }
  void release(Req* r) {
    if (!r->blocks.empty()) running -= 1;
    for (int32_t b : r->blocks) free_pool.push(b);
    r->blocks.clear();
  }
  void waitq_insert(Req* r) {  // sorted insert (admission and preemption)
    if (r->in_waitq) {
      waitq_stale -= 1;  // a stale entry becomes valid again
      return;
    }
    r->in_waitq = true;
    if (waitq.empty() || !by_arrival(r, waitq.back()))
      waitq.push_back(r);
    else
      waitq.insert(std::upper_bound(waitq.begin(), waitq.end(), r, by_arrival), r);
  }
  void compact() {
    if (waitq_stale > 32 && waitq_stale * 2 > waitq.size()) {
      size_t j = 0;
      for (Req* r : waitq) {
        if (r->waiting())
          waitq[j++] = r;
        else
          r->in_waitq = false;
      }
      waitq.resize(j);
      waitq_stale = 0;
    }
    if (active_finished > 64 && active_finished * 2 > active.size()) {
      active.erase(std::remove_if(active.begin(), active.end(), [](Req* r) { return r->finished; }), active.end());
      active_finished = 0;
    }
  }
};

namespace {

int32_t throttle_prefill(const gllm_sched_cfg& c, int64_t wp, int64_t free_blocks) {
  const int64_t n = c.num_blocks, num = c.kvthresh_num, den = c.kvthresh_den;
  if (wp == 0 || free_blocks * den < num * n) return 0;  // KV_free < KV_thresh: suspend (L165)
  int64_t cap = ((int64_t)c.maxp * (free_blocks * den - num * n)) / (n * (den - num));
  int64_t p;
  if (c.policy == GLLM_POLICY_NO_WT)
    p = cap;                                             // R19: Eq.3 without the #WP/#T term
  else if (c.policy == GLLM_POLICY_NO_UT)
    p = std::min<int64_t>(wp / c.iterp, c.maxp);         // R20: Eq.1 (threshold kept)
  else
    p = std::min(wp / c.iterp, cap);                     // Eq.3 inner min (WT vs UT)
  p = std::max(p, (int64_t)c.minp);                      // Eq.3 outer max (#MinP)
  return (int32_t)std::min(p, wp);                       // R11: cannot exceed #WP
}

// R21 (policy 4, L354): token-equivalent cost of a chunk of c tokens at offset s -- its linear
// work (c) plus its causal attention pairs c*s + c(c+1)/2 in units of attn_pairs_per_token.
int64_t chunk_cost(int64_t s, int64_t c, int64_t a) { return c + (c * s + c * (c + 1) / 2) / a; }

// largest c in [0, cmax] with chunk_cost(s, c) <= budget (chunk_cost is increasing in c)
int64_t max_chunk_within(int64_t s, int64_t cmax, int64_t budget, int64_t a) {
  int64_t lo = 0, hi = std::min(cmax, budget);  // cost >= c
  while (lo < hi) {
    const int64_t mid = lo + (hi - lo + 1) / 2;
    if (chunk_cost(s, mid, a) <= budget)
      lo = mid;
    else
      hi = mid - 1;
  }
  return lo;
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
  if (c->policy < GLLM_POLICY_THROTTLE || c->policy > GLLM_POLICY_CTX)
    return gllm::set_error(GLLM_EINVAL, "unknown policy %d", c->policy);
  if (c->policy == GLLM_POLICY_CTX && c->attn_pairs_per_token < 1)
    return gllm::set_error(GLLM_EINVAL, "context-aware policy: attn_pairs_per_token must be >= 1");
  return GLLM_OK;
}

// R1-R3: apply batch b's results; requests that become ready enter readyq in (arrival, id) order.
void retire(gllm_sched* s, BatchStore& b) {
  std::vector<Req*> touched;
  touched.reserve(b.chunks.size() + b.decodes.size());
  for (auto& c : b.chunks) {
    Req* r = c.r;
    r->done_prompt += c.len;
    r->inflight -= 1;
    if (r->done_prompt == r->prefill_len) {  // prompt completes: first output token (R2)
      r->gen += 1;
      r->ready_tick = s->tick;
      s->rd += 1;
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
  struct Key {  // sort keys held by value: no pointer chasing inside the sort
    int64_t arr, id;
    Req* r;
  };
  std::vector<Key> ready;
  ready.reserve(touched.size());
  for (Req* r : touched) {
    if (r->finished) continue;
    if (r->gen >= r->output_len) {  // fixed output length (R3)
      r->finished = true;
      s->rd -= 1;  // every finishing request has its prompt done (gen >= 1)
      s->release(r);
      s->finished += 1;
      s->active_finished += 1;
    } else if (r->decode_phase() && r->inflight == 0 && r->ready_tick == s->tick) {
      ready.push_back({r->arrival, r->id, r});
    }
  }
  std::sort(ready.begin(), ready.end(),
            [](const Key& a, const Key& b) { return a.arr != b.arr ? a.arr < b.arr : a.id < b.id; });
  for (const Key& kk : ready) s->readyq.push_back(kk.r);  // ready_tick == tick >= every queued entry
}

// R14: free the victim's blocks and return it to the waiting queue for recompute.
void preempt(gllm_sched* s, Req* v) {
  if (v->decode_phase()) {
    s->rd -= 1;
    auto it = std::find(s->readyq.begin(), s->readyq.end(), v);
    if (it != s->readyq.end()) s->readyq.erase(it);
  }
  s->wp -= v->prefill_len - v->sched_prompt;
  // a victim still waiting (partially prefilled, not in flight) keeps its valid queue entry; a
  // decode-phase victim's entry (if any) is stale and waitq_insert re-validates it
  const bool valid_entry = v->in_waitq && v->waiting();
  s->release(v);
  v->prefill_len = v->orig_len + v->gen;
  v->sched_prompt = v->done_prompt = 0;
  s->wp += v->prefill_len;
  if (!valid_entry) s->waitq_insert(v);
  s->preemptions += 1;
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
  Req* p = r.get();
  s->active.push_back(p);
  s->admitted_total += 1;
  s->storage.push_back(std::move(r));
  if (p->output_len > p->gen) {
    s->rd += 1;
    s->readyq.insert(std::upper_bound(s->readyq.begin(), s->readyq.end(), p, by_ready), p);
  }
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
    if (s->spare.size() < 4) s->spare.push_back(std::move(it->second));
    s->inflight.erase(it);
  }
  // 2. admit arrivals (R4)
  if (s->pending_dirty) {
    std::stable_sort(s->pending.begin() + s->next_arrival, s->pending.end(), by_arrival);
    s->pending_dirty = false;
  }
  while (s->next_arrival < s->pending.size() && s->pending[s->next_arrival]->arrival <= k) {
    Req* r = s->pending[s->next_arrival++];
    s->active.push_back(r);
    s->admitted_total += 1;
    s->wp += r->prefill_len;
    s->waitq_insert(r);
  }
  s->compact();
  // 3. statistics (R5), maintained incrementally
  const int64_t rd = s->rd, wp = s->wp;
  const int64_t free0 = (int64_t)s->free_pool.size();
  BatchStore b;
  if (!s->spare.empty()) {  // reuse a retired batch's buffers (no page faults on large tables)
    b = std::move(s->spare.back());
    s->spare.pop_back();
    // (block_table keeps its size: the resize below then only initialises growth)
    for (auto* v : {&b.token_ids, &b.positions, &b.slots, &b.cu_q, &b.kv_len, &b.samples, &b.sampled}) v->clear();
    b.chunks.clear();
    b.decodes.clear();
    b.seq_ids.clear();
    b.preempted.clear();
    b.allocs.clear();
  }
  b.tick = k;
  auto& allocs = b.allocs;
  auto& preempted = b.preempted;
  // 4. decode selection (Eq.4; R6-R9; R14): the first min(#D, |ready|) of the ready FIFO
  const int32_t d_cnt = cfg.policy == GLLM_POLICY_SARATHI ? (int32_t)rd : throttle_decode(cfg, rd);
  const size_t n_try = std::min<size_t>((size_t)d_cnt, s->readyq.size());
  std::vector<Req*> cand(s->readyq.begin(), s->readyq.begin() + n_try);
  s->readyq.erase(s->readyq.begin(), s->readyq.begin() + n_try);
  std::vector<Req*> skipped;  // no block and no victim: stays ready, keeps its place
  b.decodes.reserve(n_try);
  for (Req* r : cand) {
    if (!r->decode_phase()) continue;  // preempted earlier this tick
    const int32_t pos = r->orig_len + r->gen - 1;
    if ((int64_t)r->blocks.size() * bs <= pos) {
      if (s->free_pool.empty()) {
        // victim: latest (arrival, id) running request, not in flight, not selected (R14)
        Req* victim = nullptr;
        for (Req* c : s->active) {
          if (c->finished || c->blocks.empty() || c->inflight != 0 || c == r || c->sel_tick == k) continue;
          if (!victim || by_arrival(victim, c)) victim = c;
        }
        if (!victim) {
          skipped.push_back(r);
          continue;
        }
        preempt(s, victim);
        preempted.push_back(victim->id);
      }
      s->alloc(r, &allocs);
    }
    b.decodes.push_back({r, pos});
    r->sel_tick = k;
  }
  for (auto i = skipped.rbegin(); i != skipped.rend(); ++i) s->readyq.push_front(*i);
  // 5. prefill count (Eq.3 + L165; R10-R12)
  int32_t p_cnt;
  if (cfg.policy == GLLM_POLICY_SARATHI)
    p_cnt = (int32_t)std::min<int64_t>(std::max<int64_t>(cfg.token_budget - (int64_t)b.decodes.size(), 0), wp);
  else
    p_cnt = throttle_prefill(cfg, wp, free0);
  // 6. prefill selection, FCFS with CPP (R13)
  int64_t p_left = p_cnt, p_tokens = 0;
  const bool ctx = cfg.policy == GLLM_POLICY_CTX;
  for (size_t wi = 0; wi < s->waitq.size() && p_left > 0; ++wi) {
    Req* r = s->waitq[wi];
    if (!r->waiting()) continue;  // stale entry
    const bool fresh = r->blocks.empty() && r->sched_prompt == 0;
    if (fresh && s->running >= cfg.max_seqs) continue;
    const int64_t remaining = r->prefill_len - r->sched_prompt;
    const int64_t capacity = ((int64_t)r->blocks.size() + (int64_t)s->free_pool.size()) * bs - r->sched_prompt;
    int64_t c, cost;
    if (ctx) {  // R21: the chunk's token-equivalent cost (linear + causal attention) fits the budget
      c = max_chunk_within(r->sched_prompt, std::min(remaining, capacity), p_left, cfg.attn_pairs_per_token);
      if (c == 0 && b.chunks.empty() && capacity > 0) c = 1;  // progress: one token at least
      if (c <= 0) break;
      cost = chunk_cost(r->sched_prompt, c, cfg.attn_pairs_per_token);
    } else {
      c = std::min(std::min(remaining, p_left), capacity);
      if (c <= 0) break;
      cost = c;
    }
    const int64_t need = ceil_div(r->sched_prompt + c, bs) - (int64_t)r->blocks.size();
    for (int64_t j = 0; j < need; ++j) s->alloc(r, &allocs);
    b.chunks.push_back({r, r->sched_prompt, (int32_t)c, r->sched_prompt + c == r->prefill_len});
    r->sched_prompt += (int32_t)c;
    s->wp -= c;
    if (!r->waiting()) s->waitq_stale += 1;
    p_left = std::max<int64_t>(p_left - cost, 0);
    p_tokens += c;
    if (c < remaining) break;  // cut by the budget (then p_left is spent) or by KV capacity (R13)
  }
  // 7. layout (R15): prefill chunks, then decodes
  b.P = p_cnt;
  b.D = d_cnt;
  const size_t S = b.chunks.size() + b.decodes.size();
  const size_t T = (size_t)p_tokens + b.decodes.size();
  b.token_ids.reserve(T);
  b.positions.reserve(T);
  b.slots.reserve(T);
  b.cu_q.reserve(S + 1);
  b.kv_len.reserve(S);
  b.seq_ids.reserve(S);
  b.samples.reserve(S);
  b.cu_q.push_back(0);
  std::vector<const Req*> rows_req;
  std::vector<int32_t> rows_n;
  rows_req.reserve(S);
  rows_n.reserve(S);
  for (auto& c : b.chunks) {
    const size_t t0 = b.token_ids.size();
    b.token_ids.insert(b.token_ids.end(), c.r->ids.begin() + c.start, c.r->ids.begin() + c.start + c.len);
    b.positions.resize(t0 + c.len);
    b.slots.resize(t0 + c.len);
    int32_t* pos = b.positions.data() + t0;
    int32_t* slot = b.slots.data() + t0;
    for (int32_t p = c.start, blk = c.start / bs, off = c.start % bs; p < c.start + c.len; ++p) {
      *pos++ = p;
      *slot++ = c.r->blocks[blk] * bs + off;  // O2: slot = bt[pos / bs] * bs + pos % bs
      if (++off == bs) {
        off = 0;
        ++blk;
      }
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
  b.block_table.resize(rows_req.size() * (size_t)b.maxblk);
  for (size_t i = 0; i < rows_req.size(); ++i) {  // one pass: blocks, then -1 padding
    int32_t* row = b.block_table.data() + i * b.maxblk;
    std::memcpy(row, rows_req[i]->blocks.data(), rows_n[i] * sizeof(int32_t));
    std::fill(row + rows_n[i], row + b.maxblk, -1);
  }
  b.rd = rd;
  b.wp = wp;
  b.free0 = free0;
  b.free1 = (int64_t)s->free_pool.size();
  s->last_tick = k;

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
  return s->next_arrival >= s->pending.size() && s->finished == s->admitted_total ? 1 : 0;
}

int gllm_sched_stats(const gllm_sched* s, int64_t* out6) {
  if (!s || !out6) return gllm::set_error(GLLM_EINVAL, "null argument");
  out6[0] = s->tick;
  out6[1] = s->running;
  out6[2] = (int64_t)s->free_pool.size();
  out6[3] = s->preemptions;
  out6[4] = s->finished;
  out6[5] = s->admitted_total;
  return GLLM_OK;
}

int gllm_sched_seq_blocks(const gllm_sched* s, int64_t req_id, int32_t* out, int32_t cap, int32_t* n) {
  GLLM_TRY_BEGIN
  if (!s || !n || (cap > 0 && !out)) return gllm::set_error(GLLM_EINVAL, "null argument");
  for (const auto& r : s->storage) {
    if (r->id != req_id) continue;
    if (r->finished) break;
    *n = (int32_t)r->blocks.size();
    if (*n > cap) return gllm::set_error(GLLM_EINVAL, "seq_blocks: cap %d < %d blocks", cap, *n);
    std::memcpy(out, r->blocks.data(), r->blocks.size() * sizeof(int32_t));
    return GLLM_OK;
  }
  return gllm::set_error(GLLM_EINVAL, "seq_blocks: request %lld not running", (long long)req_id);
  GLLM_TRY_END
}

int gllm_sched_trace(gllm_sched* s, void* buf, size_t cap, size_t* used) {
  GLLM_TRY_BEGIN
  if (!s || !used) return gllm::set_error(GLLM_EINVAL, "null argument");
  auto it = s->inflight.find(s->last_tick);
  if (it == s->inflight.end()) return gllm::set_error(GLLM_ESTATE, "no batch built since the last retire");
  const BatchStore& b = it->second;
  // canonical trace (== oracle.scheduler.trace_bytes)
  std::vector<int64_t> t;
  const int64_t T = (int64_t)b.token_ids.size();
  t.insert(t.end(), {b.tick, (int64_t)b.P, (int64_t)b.D, b.rd, b.wp, b.free0, b.free1, (int64_t)b.chunks.size(),
                     (int64_t)b.decodes.size(), (int64_t)b.preempted.size(), (int64_t)b.allocs.size(), T,
                     (int64_t)b.samples.size()});
  for (auto& c : b.chunks) t.insert(t.end(), {c.r->id, (int64_t)c.start, (int64_t)c.len});
  for (auto& d : b.decodes) t.insert(t.end(), {d.r->id, (int64_t)d.pos});
  for (int64_t v : b.preempted) t.push_back(v);
  for (auto& a : b.allocs) t.insert(t.end(), {a.first, (int64_t)a.second});
  for (int32_t v : b.slots) t.push_back(v);
  for (int32_t v : b.samples) t.push_back(v);
  const size_t n = t.size() * sizeof(int64_t);
  *used = n;
  if (cap < n || (!buf && n)) return gllm::set_error(GLLM_EINVAL, "trace buffer too small (%zu < %zu)", cap, n);
  if (n) std::memcpy(buf, t.data(), n);
  return GLLM_OK;
  GLLM_TRY_END
}

}  // extern "C"
