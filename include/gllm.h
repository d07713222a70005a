/* gllm.h -- C ABI of the B200-native per-stage mixed-batch forward of gLLM
 * (Guo et al., "gLLM: Global Balanced Pipeline Parallelism Systems for
 * Distributed LLMs Serving with Token Throttling", SC'25).
 * Citations "Lnnn" are line numbers of /root/reference/PAPER.md.
 *
 * Conventions
 *   - Every call returns int: 0 = GLLM_OK, > 0 = benign status, < 0 = error.
 *     gllm_last_error() returns the thread-local message of the last error.
 *     No C++ exception crosses the ABI; nothing aborts or prints.
 *   - "host" pointers are ordinary CPU memory; "device" pointers are CUDA
 *     global memory of the stage's device.  Buffers passed in are owned by the
 *     caller unless stated otherwise; the library never frees them.
 *   - No torch types appear here; PyTorch only allocates hidden buffers /
 *     streams and exchanges the NCCL unique id (north_star).
 */
#ifndef GLLM_H
#define GLLM_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define GLLM_API __attribute__((visibility("default")))
#else
#define GLLM_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

enum {
  GLLM_OK = 0,
  GLLM_EMPTY = 1,      /* tick had nothing to schedule (R16) */
  GLLM_EINVAL = -1,    /* argument / batch validation failed */
  GLLM_ENOMEM = -2,    /* device or host allocation failed */
  GLLM_ECUDA = -3,     /* CUDA runtime error (message has cudaGetErrorString) */
  GLLM_ENCCL = -4,     /* NCCL error */
  GLLM_ESTATE = -5     /* call out of order (e.g. retire of an unknown tick) */
};

GLLM_API const char* gllm_last_error(void);
/* Library build tag: "gllm-b200 sm_100a <git-less version>". */
GLLM_API const char* gllm_version(void);

/* ------------------------------------------------------------------------ */
/* Model (the decoder-only transformer of L73 §2.1; Llama / Qwen2 shapes of  */
/* the paper's evaluation, L218/L224).                                        */
/* ------------------------------------------------------------------------ */
typedef struct {
  int32_t n_layers, hidden, n_heads, n_kv_heads, head_dim, intermediate, vocab;
  float rms_eps, rope_theta;
  int32_t qkv_bias;      /* 1 = Qwen2-style q/k/v biases */
  uint64_t weight_seed;  /* O4 counter-based weight generator seed */
} gllm_model_cfg;

/* ------------------------------------------------------------------------ */
/* Scheduler: Token Throttling (L145-L183 §3.1-3.2) + paged-KV block manager */
/* (L136 Fig.6).  Host-only, deterministic, single-threaded per object. */
/* ------------------------------------------------------------------------ */
/* build_batch policies (gllm_sched_cfg.policy) */
enum { GLLM_POLICY_THROTTLE = 0, GLLM_POLICY_SARATHI = 1, GLLM_POLICY_NO_WT = 2, GLLM_POLICY_NO_UT = 3,
       GLLM_POLICY_CTX = 4 };

typedef struct {
  int32_t iterp;          /* #T  (Eq.1/Eq.3; default 8, L248) */
  int32_t maxp, minp;     /* #MaxP, #MinP (L151; 2048 / 32, L248) */
  int32_t kvthresh_num;   /* KV_thresh = num/den (L165; 0.05 = 1/20, L248); 0 <= num < den */
  int32_t kvthresh_den;
  int32_t pp_depth;       /* #PP_depth (Eq.4) = max micro-batches in flight (L179) */
  int32_t num_blocks;     /* N, KV blocks shared by all stages (L136) */
  int32_t block_size;     /* tokens per KV block (16) */
  int32_t max_seqs;       /* max running sequences (1024, L575) */
  int32_t policy;         /* GLLM_POLICY_*: 0 = Token Throttling (Eq.3 + threshold, Eq.4);
                             1 = Sarathi-Serve (every ready decode, prefill to token_budget; "w/ CK", L310);
                             2 = ablation "w/o WT" (Eq.3 without the #WP/#T term, L308);
                             3 = ablation "w/o UT" (Eq.1 + the L165 threshold, L308).
                             Policies 2-3 keep Eq.4 for decodes (§4.5, Fig. 15).
                             4 = context-aware Token Throttling (the paper's future work, L354;
                             reading R21 in DESIGN.md): #P of Eq.3 is a budget in token
                             equivalents and a chunk of c tokens at offset s costs
                             c + floor((c*s + c*(c+1)/2) / attn_pairs_per_token). */
  int32_t token_budget;   /* Sarathi only (2048, L248) */
  int32_t attn_pairs_per_token; /* policy 4 only: causal (query, key) pairs whose attention costs
                             as much as one token's linear layers (>= 1) */
} gllm_sched_cfg;

typedef struct gllm_sched gllm_sched;

/* Creates a scheduler.  EINVAL on non-positive sizes or kvthresh outside [0,1). */
GLLM_API int gllm_sched_create(const gllm_sched_cfg* cfg, gllm_sched** out);
GLLM_API int gllm_sched_free(gllm_sched* s);

/* Queues a request arriving at `arrival_tick` (reading R4: arrivals in ticks).
 * token_ids: host, prompt_len + output_len - 1 ids (prompt, then the
 * teacher-forced outputs t1..t_{out-1}, R17); copied.  EINVAL on
 * prompt_len < 1, output_len < 1 or a duplicate req_id. */
GLLM_API int gllm_sched_add_request(gllm_sched* s, int64_t req_id, int64_t arrival_tick,
                           int32_t prompt_len, int32_t output_len, const int32_t* token_ids);

/* Adds a sequence already in decode (warm start, C4): context_len tokens are
 * cached (blocks allocated now, lowest first) and remaining_out decodes follow.
 * token_ids: host, context_len + remaining_out ids; copied.  ENOMEM if the
 * pool cannot hold the context. */
GLLM_API int gllm_sched_add_warm(gllm_sched* s, int64_t req_id, int32_t context_len,
                        int32_t remaining_out, const int32_t* token_ids);

/* Pure Eq.3 + L165 threshold (P) and Eq.4 (D) in exact integer arithmetic
 * (readings R6, R10, R11):
 *   P = 0 if wp == 0 or free*den < num*N, else
 *   P = min(max(min(wp / iterp, MaxP*(free*den - num*N) / (N*(den-num))), MinP), wp)
 *   D = ceil(rd / pp_depth)                              (all divisions floor) */
GLLM_API int gllm_throttle_counts(const gllm_sched_cfg* cfg, int64_t wp, int64_t rd, int32_t free_blocks,
                         int32_t* P, int32_t* D);

/* One scheduled micro-batch (D3/D4 of SURVEY §2.3).  Layout (R15): prefill
 * chunks first (selection order), then decode tokens.  All arrays are host
 * memory owned by the scheduler and valid until gllm_retire_batch(tick). */
typedef struct {
  int64_t tick;
  int32_t P, D;                 /* counts computed by Eq.3 / Eq.4 this tick */
  int32_t num_prefill_tokens, num_decode_tokens, num_tokens;
  int32_t num_seqs, num_prefill_seqs, max_blocks_per_seq, num_samples;
  const int32_t* token_ids;     /* [num_tokens] */
  const int32_t* positions;     /* [num_tokens] absolute positions */
  const int32_t* slot_mapping;  /* [num_tokens] slot = bt[pos/bs]*bs + pos%bs (O2) */
  const int32_t* cu_q;          /* [num_seqs+1] token offsets of each sequence */
  const int32_t* kv_len;        /* [num_seqs] keys visible to the sequence's last token */
  const int32_t* block_table;   /* [num_seqs * max_blocks_per_seq], -1 padded */
  const int32_t* sample_token_idx; /* [num_samples] rows whose next token is sampled */
  const int64_t* seq_req_ids;   /* [num_seqs] */
} gllm_batch_desc;

/* Builds the micro-batch of the current tick k and advances the tick:
 * retires batch k - pp_depth first (R1), admits arrivals, computes the global
 * statistics #WP, #RD, KV_free (L151, L161, L183), throttles (Eq.3, Eq.4),
 * selects decodes then prefill chunks, allocates blocks (decode first, lowest
 * free block first) and fills *out.  Returns GLLM_EMPTY (with *out valid,
 * num_tokens == 0) for a tick with nothing scheduled; the tick still occupies
 * an in-flight slot (R16). */
GLLM_API int gllm_build_batch(gllm_sched* s, gllm_batch_desc* out);

/* Optionally records the sampled ids of `tick` early (the automatic retire in
 * build_batch k+pp_depth then applies them).  sampled_ids: host
 * [num_samples] or NULL.  ESTATE if tick is not in flight. */
GLLM_API int gllm_retire_batch(gllm_sched* s, int64_t tick, const int32_t* sampled_ids);

/* 1 when every request has finished and no arrival is pending. */
GLLM_API int gllm_sched_done(const gllm_sched* s);

/* Scheduler statistics: [0] tick, [1] running requests, [2] free blocks,
 * [3] preemptions so far, [4] finished requests, [5] requests admitted. */
GLLM_API int gllm_sched_stats(const gllm_sched* s, int64_t* out6);

/* Block ids of a running (not finished) request, in position order: *n receives the count;
 * out: host int32 [cap].  EINVAL if the request is unknown or finished, or cap < *n. */
GLLM_API int gllm_sched_seq_blocks(const gllm_sched* s, int64_t req_id, int32_t* out, int32_t cap, int32_t* n);

/* Canonical little-endian int64 trace of the LAST built tick (layout in
 * DESIGN.md §3; identical to oracle.scheduler.trace_bytes).  *used receives
 * the byte count; EINVAL if cap is too small (then *used is the size needed). */
GLLM_API int gllm_sched_trace(gllm_sched* s, void* buf, size_t cap, size_t* used);

/* ------------------------------------------------------------------------ */
/* Stage: one pipeline stage's layers on one GPU (P1, L90-L92, L198).         */
/* ------------------------------------------------------------------------ */
typedef struct gllm_stage gllm_stage;

/* init_stage(layers, kv_blocks): allocates on `device` the bf16 weights of
 * layers [layer_begin, layer_end) (+ embedding if layer_begin == 0, + final
 * norm and LM head if layer_end == n_layers), fills them with the O4
 * generator on the GPU, allocates the paged KV cache (kv_blocks x block_size
 * tokens for every local layer) and workspaces for up to max_tokens tokens and
 * max_seqs sequences per micro-batch.  EINVAL for inconsistent shapes
 * (head_dim != 128 and != 64, hidden % 64, intermediate % 128, ...), ENOMEM
 * when HBM does not fit.
 * Restriction: every RMSNorm gain is 1 (the O4 weights).  The library has no
 * gain input: the fused norm scales GEMM rows by 1/rms(x) and would need a gain folded into the
 * columns of W_qkv / W_gate_up (W' = W diag(g)), which O4's g = 1 makes the identity. */
GLLM_API int gllm_init_stage(const gllm_model_cfg* cfg, int32_t layer_begin, int32_t layer_end,
                    int32_t kv_blocks, int32_t block_size, int32_t max_tokens,
                    int32_t max_seqs, int32_t device, gllm_stage** out);
GLLM_API int gllm_free_stage(gllm_stage* st);

/* stage_forward(batch_desc, hidden_in, hidden_out): enqueues the whole stage
 * forward on `stream` (a cudaStream_t, NULL = the legacy default stream) and
 * returns immediately.  The desc is validated (T <= max_tokens, S <= max_seqs,
 * block ids < kv_blocks, positions < kv_len -> EINVAL) and snapshotted into
 * stage-owned pinned staging before return, so the caller may reuse it.
 *   hidden_in:   device fp32 [num_tokens, hidden]; ignored (may be NULL) on stage 0.
 *   hidden_out:  device fp32 [num_tokens, hidden] residual after the last local
 *                layer; may be NULL on the last stage; may equal hidden_in.
 *   sampled_out: device int32 [num_samples] greedy ids (last stage only; may be NULL).
 * Async CUDA errors surface on the next call or on gllm_stage_sync. */
GLLM_API int gllm_stage_forward(gllm_stage* st, const gllm_batch_desc* desc, const void* hidden_in,
                       void* hidden_out, int32_t* sampled_out, void* stream);

/* Two-phase form of stage_forward, after the paper's dual-phase transmission
 * (L204): prepare() validates the desc, builds the attention work lists and
 * copies all metadata to a stage-owned device slot on `stream` as soon as the
 * schedule is known; forward_prepared() later launches the layers once the
 * activations arrive (it waits on the slot's copy event, any stream).  The
 * handle stays valid until gllm_stage_release(); a slot is only reused after
 * its last forward completed.  Same errors as gllm_stage_forward. */
GLLM_API int gllm_stage_prepare(gllm_stage* st, const gllm_batch_desc* desc, void* stream, int32_t* handle);
GLLM_API int gllm_stage_forward_prepared(gllm_stage* st, int32_t handle, const void* hidden_in, void* hidden_out,
                                         int32_t* sampled_out, void* stream);
GLLM_API int gllm_stage_release(gllm_stage* st, int32_t handle);

/* Pipeline hand-off (a12; activations over NCCL, L222).  comm_init joins an
 * NCCL communicator of `world` ranks (unique_id: 128 bytes from ncclGetUniqueId,
 * exchanged by the caller).  send/recv move num_tokens x hidden fp32 rows of a
 * device buffer to/from rank dst/src on `stream`. */
GLLM_API int gllm_get_unique_id(void* out128);
GLLM_API int gllm_comm_init(gllm_stage* st, const void* nccl_unique_id, int32_t rank, int32_t world);
/* The communicator's size and this stage's rank in it (ncclCommCount / ncclCommUserRank). */
GLLM_API int gllm_comm_size(gllm_stage* st, int32_t* nranks, int32_t* rank);
GLLM_API int gllm_send_hidden(gllm_stage* st, const void* buf, int32_t num_tokens, int32_t dst, void* stream);
GLLM_API int gllm_recv_hidden(gllm_stage* st, void* buf, int32_t num_tokens, int32_t src, void* stream);
GLLM_API int gllm_stage_sync(gllm_stage* st);

/* Fused stage hand-off over peer memory (a12; PAPER.md L198, L204,
 * L222): instead of an NCCL send/recv, stage s writes its output residual straight into a
 * receive slot in stage s+1's device memory (NVLink peer stores, CUDA IPC mapping; on one GPU
 * two processes share the device) from the last layer's residual-add GEMM epilogue, and raises
 * the slot's flag with a system-scope release store after its last kernel.  Stage s+1's stream
 * waits on that flag (cuStreamWaitValue32) and reads the slot as hidden_in.
 * Slot reuse is flow-controlled, independent of host timing: micro-batch `tick` uses slot
 * tick % depth; the receiver's stage-entry kernel (the one pass that reads the slot) releases a
 * credit for the slot (credit = tick + 1, system-scope release store from its last CTA into the
 * sender's memory) and the sender's stream waits for credit >= tick - depth + 1 before it
 * enqueues the forward that overwrites the slot.  Both waits are on local memory; both signals
 * are remote stores.  Set-up order: receiver gllm_peer_ring_create -> sender gllm_peer_ring_open
 * (returns the credit handle) -> receiver gllm_peer_credit_open.  The credits are mandatory: a
 * sender whose receiver never opened them stalls at tick `depth`.
 * Errors: EINVAL on bad arguments or a shape mismatch, ESTATE on the wrong stage role or a ring
 * already created/opened, ECUDA on CUDA/IPC failures. */
#define GLLM_PEER_HANDLE_BYTES 128
/* Receiver (not the first stage): allocates depth (1..64) slots of [max_tokens, hidden] fp32 plus
 * depth 32-bit flags (zero) in one exportable allocation; writes the IPC handle (caller-owned, 128 B). */
GLLM_API int gllm_peer_ring_create(gllm_stage* st, int32_t depth, void* handle_out);
/* Sender (not the last stage): maps the receiver's ring from its handle and allocates the slot
 * credits (depth 32-bit flags, zero) in its own memory; writes their IPC handle to
 * credit_handle_out (caller-owned, 128 B).  The receiver must live in another process (CUDA IPC
 * handles cannot be opened by the exporting process): ECUDA. */
GLLM_API int gllm_peer_ring_open(gllm_stage* st, const void* handle, void* credit_handle_out);
/* Receiver: maps the sender's slot credits (handle from gllm_peer_ring_open). */
GLLM_API int gllm_peer_credit_open(gllm_stage* st, const void* credit_handle);
/* Sender: the forward of a prepared batch with its output delivered to the receiver's slot for
 * `tick` (hidden_out is the slot); waits on the slot's credit first (tick >= depth); flag =
 * tick + 1 after the forward's last kernel. */
GLLM_API int gllm_stage_forward_prepared_peer(gllm_stage* st, int32_t handle, const void* hidden_in,
                                              int64_t tick, void* stream);
/* Receiver: enqueues on `stream` a wait for the sender's release of `tick`; *slot_out = the
 * device pointer of that slot.  The next forward on this stage whose hidden_in is that slot reads
 * it in its first kernel and releases the slot's credit. */
GLLM_API int gllm_peer_ring_recv(gllm_stage* st, int64_t tick, void* stream, void** slot_out);

/* Introspection for parity tests (host outputs, synchronous). */
/* Copies element range [row0, row0+nrows) x all columns of a logical weight
 * ("wq","wk","wv","wo","wg","wu","wd","bq","bk","bv","embed","lm_head") of
 * `layer` as fp32 into host `out`. */
GLLM_API int gllm_stage_read_weight(gllm_stage* st, int32_t layer, const char* name, int64_t row0,
                           int64_t nrows, float* out);
/* Reads K and V of `n` cache slots of local `layer` as fp32 host [n, n_kv_heads, head_dim]. */
GLLM_API int gllm_stage_read_kv(gllm_stage* st, int32_t layer, const int32_t* slots, int32_t n,
                       float* k_out, float* v_out);
/* Device slot mapping produced by the last stage_forward, host int32 [num_tokens]. */
GLLM_API int gllm_stage_read_slots(gllm_stage* st, int32_t* out, int32_t n);
/* Warm start (C4's warm decode set): writes the cached K and V of
 * positions [0, context_lens[i]) of warm request req_ids[i], for every local layer, through row i of
 * block_table (host int32 [n_seqs * max_blocks], the blocks the scheduler gave the sequence, see
 * gllm_sched_seq_blocks).  Values follow O4 with the model's weight seed: K (V) of request r,
 * position p, layer l, kv head h, dim j is element ((r * 2^17 + p) * n_kv_heads + h) * head_dim + j
 * of tensor 0xEE0000 + 2l (+1), scale sqrt(3), rounded to bf16 (oracle.weights.warm_kv holds the same
 * values).  Host arrays are copied; synchronous.  EINVAL for contexts outside [1, 2^17], request ids
 * outside the 40-bit index range, or block ids >= kv_blocks. */
GLLM_API int gllm_stage_fill_warm_kv(gllm_stage* st, int32_t n_seqs, const int64_t* req_ids,
                                     const int32_t* context_lens, const int32_t* block_table, int32_t max_blocks);

/* on = 1: every later forward of this stage uses GEMM schedules with a fixed reduction order (whole
 * tiles or cluster split-K instead of stream-K / hybrid tails, whose fp32 atomic adds make the
 * last bits depend on arrival order; RMSNorm row statistics from the standalone pass instead of
 * the epilogue's per-tile atomic sum).  Results are then bitwise reproducible run to run (the
 * attention kernels always are).  Costs a few % at shapes that would take stream-K.  Default 0. */
GLLM_API int gllm_stage_set_deterministic(gllm_stage* st, int32_t on);

/* Timing of the forwards since the previous call, from CUDA events recorded on each forward's own
 * stream around each launch (enabled by gllm_stage_set_profiling(st, 1)).  on = 2 also runs the
 * prefill and decode attention kernels in series instead of on two concurrent streams, so that each
 * one's events bracket that kernel alone (an attribution pass; the forward's results are the same).
 * out[n] receives milliseconds per category (synchronises on the events):
 *   [0] whole forward  [1] QKV GEMM  [2] O GEMM  [3] gate_up GEMM  [4] down GEMM
 *   [5] prefill attention  [6] decode attention  [7] RoPE+KV append  [8] RMSNorm
 *   [9] final norm + LM head + argmax  [10] other (prep, embedding) */
GLLM_API int gllm_stage_set_profiling(gllm_stage* st, int32_t on);
GLLM_API int gllm_stage_last_timing(gllm_stage* st, float* out, int32_t n);
/* Number of kernels the last stage_forward launched. */
GLLM_API int gllm_stage_last_launches(gllm_stage* st, int32_t* out);

#ifdef __cplusplus
}
#endif
#endif /* GLLM_H */
