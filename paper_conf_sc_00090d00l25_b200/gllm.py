"""Thin ctypes binding of libgllm.so (include/gllm.h).  Argument marshalling only:
every step of the hot path runs in the library's CUDA kernels / C++ scheduler.

Names follow the C ABI without the `gllm_` prefix: `sched_create`,
`build_batch`, `retire_batch`, `throttle_counts`, `init_stage`,
`stage_forward`, `send_hidden`, `recv_hidden`, ...  There is no fallback: if the
shared library is missing, `lib()` raises.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GLLM_LIB") or os.path.join(_HERE, "libgllm.so")  # GLLM_LIB: measurement builds

GLLM_OK, GLLM_EMPTY = 0, 1
ERRORS = {-1: "EINVAL", -2: "ENOMEM", -3: "ECUDA", -4: "ENCCL", -5: "ESTATE"}

TIMING_NAMES = ["total", "qkv_gemm", "o_gemm", "gate_up_gemm", "down_gemm", "prefill_attn", "decode_attn",
                "rope_kv_append", "rmsnorm", "lm_head", "other", "attention_span"]


class GllmError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"{ERRORS.get(code, code)}: {msg}")
        self.code = code


class ModelCfg(C.Structure):
    _fields_ = [("n_layers", C.c_int32), ("hidden", C.c_int32), ("n_heads", C.c_int32),
                ("n_kv_heads", C.c_int32), ("head_dim", C.c_int32), ("intermediate", C.c_int32),
                ("vocab", C.c_int32), ("rms_eps", C.c_float), ("rope_theta", C.c_float),
                ("qkv_bias", C.c_int32), ("weight_seed", C.c_uint64)]


class SchedCfg(C.Structure):
    _fields_ = [(n, C.c_int32) for n in ("iterp", "maxp", "minp", "kvthresh_num", "kvthresh_den", "pp_depth",
                                           "num_blocks", "block_size", "max_seqs", "policy", "token_budget",
                                           "attn_pairs_per_token")]


_P32 = C.POINTER(C.c_int32)
_P64 = C.POINTER(C.c_int64)


class BatchDesc(C.Structure):
    _fields_ = [("tick", C.c_int64), ("P", C.c_int32), ("D", C.c_int32),
                ("num_prefill_tokens", C.c_int32), ("num_decode_tokens", C.c_int32), ("num_tokens", C.c_int32),
                ("num_seqs", C.c_int32), ("num_prefill_seqs", C.c_int32), ("max_blocks_per_seq", C.c_int32),
                ("num_samples", C.c_int32),
                ("token_ids", _P32), ("positions", _P32), ("slot_mapping", _P32), ("cu_q", _P32),
                ("kv_len", _P32), ("block_table", _P32), ("sample_token_idx", _P32), ("seq_req_ids", _P64)]

    def arr(self, name, n, dtype=np.int32):
        p = getattr(self, name)
        if n == 0 or not p:
            return np.zeros(0, dtype)
        return np.ctypeslib.as_array(p, shape=(n,)).copy()

    def to_numpy(self) -> dict:
        T, S = self.num_tokens, self.num_seqs
        return dict(tick=self.tick, P=self.P, D=self.D, num_tokens=T, num_seqs=S,
                    num_prefill_seqs=self.num_prefill_seqs, token_ids=self.arr("token_ids", T),
                    positions=self.arr("positions", T), slot_mapping=self.arr("slot_mapping", T),
                    cu_q=self.arr("cu_q", S + 1 if S else 0), kv_len=self.arr("kv_len", S),
                    block_table=self.arr("block_table", S * self.max_blocks_per_seq).reshape(
                        S, self.max_blocks_per_seq) if S else np.zeros((0, 0), np.int32),
                    sample_idx=self.arr("sample_token_idx", self.num_samples),
                    seq_req_ids=self.arr("seq_req_ids", S, np.int64))


_lib = None


def lib():
    """Loads libgllm.so (raises if it was not built: there is no CPU fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} missing: run `python -m paper_conf_sc_00090d00l25_b200.build`")
        L = C.CDLL(LIB_PATH)
        vp, i32, i64, u64, sz = C.c_void_p, C.c_int32, C.c_int64, C.c_uint64, C.c_size_t
        sig = {
            "gllm_last_error": ([], C.c_char_p), "gllm_version": ([], C.c_char_p),
            "gllm_sched_create": ([C.POINTER(SchedCfg), C.POINTER(vp)], C.c_int),
            "gllm_sched_free": ([vp], C.c_int),
            "gllm_sched_add_request": ([vp, i64, i64, i32, i32, _P32], C.c_int),
            "gllm_sched_add_warm": ([vp, i64, i32, i32, _P32], C.c_int),
            "gllm_throttle_counts": ([C.POINTER(SchedCfg), i64, i64, i32, _P32, _P32], C.c_int),
            "gllm_build_batch": ([vp, C.POINTER(BatchDesc)], C.c_int),
            "gllm_retire_batch": ([vp, i64, _P32], C.c_int),
            "gllm_sched_done": ([vp], C.c_int),
            "gllm_sched_stats": ([vp, _P64], C.c_int),
            "gllm_sched_trace": ([vp, vp, sz, C.POINTER(sz)], C.c_int),
            "gllm_init_stage": ([C.POINTER(ModelCfg), i32, i32, i32, i32, i32, i32, i32, C.POINTER(vp)], C.c_int),
            "gllm_free_stage": ([vp], C.c_int),
            "gllm_stage_forward": ([vp, C.POINTER(BatchDesc), vp, vp, vp, vp], C.c_int),
            "gllm_stage_prepare": ([vp, C.POINTER(BatchDesc), vp, _P32], C.c_int),
            "gllm_stage_forward_prepared": ([vp, i32, vp, vp, vp, vp], C.c_int),
            "gllm_stage_release": ([vp, i32], C.c_int),
            "gllm_get_unique_id": ([vp], C.c_int),
            "gllm_comm_init": ([vp, vp, i32, i32], C.c_int),
            "gllm_comm_size": ([vp, _P32, _P32], C.c_int),
            "gllm_send_hidden": ([vp, vp, i32, i32, vp], C.c_int),
            "gllm_recv_hidden": ([vp, vp, i32, i32, vp], C.c_int),
            "gllm_stage_sync": ([vp], C.c_int),
            "gllm_peer_ring_create": ([vp, i32, vp], C.c_int),
            "gllm_peer_ring_open": ([vp, vp, vp], C.c_int),
            "gllm_peer_credit_open": ([vp, vp], C.c_int),
            "gllm_stage_forward_prepared_peer": ([vp, i32, vp, i64, vp], C.c_int),
            "gllm_peer_ring_recv": ([vp, i64, vp, C.POINTER(C.c_void_p)], C.c_int),
            "gllm_stage_read_weight": ([vp, i32, C.c_char_p, i64, i64, C.POINTER(C.c_float)], C.c_int),
            "gllm_stage_read_kv": ([vp, i32, _P32, i32, C.POINTER(C.c_float), C.POINTER(C.c_float)], C.c_int),
            "gllm_stage_read_slots": ([vp, _P32, i32], C.c_int),
            "gllm_stage_fill_warm_kv": ([vp, i32, C.POINTER(C.c_int64), _P32, _P32, i32], C.c_int),
            "gllm_sched_seq_blocks": ([vp, i64, _P32, i32, _P32], C.c_int),
            "gllm_stage_set_profiling": ([vp, i32], C.c_int),
            "gllm_stage_set_deterministic": ([vp, i32], C.c_int),
            "gllm_stage_last_timing": ([vp, C.POINTER(C.c_float), i32], C.c_int),
            "gllm_stage_last_launches": ([vp, _P32], C.c_int),
            "gllm_op_gemm": ([vp, vp, i32, i32, i32, i32, vp, vp, vp], C.c_int),
            "gllm_op_set_gemm_variant": ([i32], C.c_int),
            "gllm_op_set_deterministic": ([i32], C.c_int),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def _check(rc):
    if rc < 0:
        raise GllmError(rc, lib().gllm_last_error().decode())
    return rc


def _p32(a):
    return a.ctypes.data_as(_P32)


def version() -> str:
    return lib().gllm_version().decode()


# ------------------------------------------------------------------ scheduler
def sched_cfg(p) -> SchedCfg:
    """SchedCfg from a workloads.SchedParams (or any object with the same fields)."""
    return SchedCfg(*(int(getattr(p, f)) for f, _ in SchedCfg._fields_))


def throttle_counts(cfg, wp: int, rd: int, free_blocks: int):
    P, D = C.c_int32(), C.c_int32()
    c = cfg if isinstance(cfg, SchedCfg) else sched_cfg(cfg)
    _check(lib().gllm_throttle_counts(C.byref(c), wp, rd, free_blocks, C.byref(P), C.byref(D)))
    return P.value, D.value


class Sched:
    """Owner of a gllm_sched*: Token Throttling + block manager (host)."""

    def __init__(self, cfg):
        self.cfg = cfg if isinstance(cfg, SchedCfg) else sched_cfg(cfg)
        h = C.c_void_p()
        _check(lib().gllm_sched_create(C.byref(self.cfg), C.byref(h)))
        self.h = h

    def close(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.gllm_sched_free(self.h)
            self.h = None

    __del__ = close

    def add_request(self, req_id, arrival_tick, prompt_len, output_len, token_ids):
        ids = np.ascontiguousarray(token_ids, dtype=np.int32)
        assert ids.shape[0] >= prompt_len + output_len - 1
        _check(lib().gllm_sched_add_request(self.h, req_id, arrival_tick, prompt_len, output_len, _p32(ids)))

    def add_warm(self, req_id, context_len, remaining_out, token_ids):
        ids = np.ascontiguousarray(token_ids, dtype=np.int32)
        _check(lib().gllm_sched_add_warm(self.h, req_id, context_len, remaining_out, _p32(ids)))

    def add_stream(self, stream):
        for w in stream.warm:
            self.add_warm(w.req_id, w.context_len, w.remaining_out, w.token_ids)
        for r in stream.requests:
            self.add_request(r.req_id, r.arrival_tick, r.prompt_len, r.output_len, r.token_ids)

    def build_batch(self) -> BatchDesc:
        d = BatchDesc()
        _check(lib().gllm_build_batch(self.h, C.byref(d)))
        return d

    def retire_batch(self, tick, sampled=None):
        if sampled is None:
            return _check(lib().gllm_retire_batch(self.h, tick, None))
        s = np.ascontiguousarray(sampled, dtype=np.int32)
        return _check(lib().gllm_retire_batch(self.h, tick, _p32(s)))

    def done(self) -> bool:
        return bool(lib().gllm_sched_done(self.h))

    def stats(self) -> dict:
        out = (C.c_int64 * 6)()
        _check(lib().gllm_sched_stats(self.h, out))
        return dict(zip(["tick", "running", "free_blocks", "preemptions", "finished", "admitted"], list(out)))

    def seq_blocks(self, req_id) -> np.ndarray:
        n = C.c_int32()
        rc = lib().gllm_sched_seq_blocks(self.h, req_id, None, 0, C.byref(n))
        out = np.zeros(max(n.value, 1), np.int32)
        if rc != 0:
            _check(lib().gllm_sched_seq_blocks(self.h, req_id, _p32(out), out.shape[0], C.byref(n)))
        return out[: n.value]

    def trace(self) -> bytes:
        used = C.c_size_t()
        rc = lib().gllm_sched_trace(self.h, None, 0, C.byref(used))
        buf = C.create_string_buffer(max(used.value, 1))
        _check(lib().gllm_sched_trace(self.h, buf, used.value, C.byref(used)))
        return buf.raw[:used.value]


def sched_create(cfg) -> Sched:
    return Sched(cfg)


# ------------------------------------------------------------------ stage
def model_cfg(m) -> ModelCfg:
    """ModelCfg from a workloads.ModelShape."""
    return ModelCfg(m.n_layers, m.hidden, m.n_heads, m.n_kv_heads, m.head_dim, m.intermediate, m.vocab,
                    m.rms_eps, m.rope_theta, int(m.qkv_bias), m.weight_seed)


def desc_from_arrays(a: dict):
    """BatchDesc pointing at numpy arrays in `a` (keeps them alive in the returned tuple)."""
    keep = {k: np.ascontiguousarray(v, dtype=np.int64 if k == "seq_req_ids" else np.int32)
            for k, v in a.items() if k in ("token_ids", "positions", "slot_mapping", "cu_q", "kv_len",
                                          "block_table", "sample_idx", "seq_req_ids")}
    d = BatchDesc()
    T = int(keep["token_ids"].shape[0])
    S = int(keep["cu_q"].shape[0]) - 1 if keep["cu_q"].shape[0] else 0
    bt = keep["block_table"].reshape(S, -1) if S else keep["block_table"].reshape(0, 0)
    keep["block_table"] = np.ascontiguousarray(bt)
    d.tick = int(a.get("tick", 0))
    d.num_tokens = T
    d.num_seqs = S
    d.num_prefill_seqs = int(a["num_prefill_seqs"])
    d.max_blocks_per_seq = int(bt.shape[1]) if S else 0
    d.num_samples = int(keep["sample_idx"].shape[0])
    d.num_prefill_tokens = int(keep["cu_q"][d.num_prefill_seqs]) if S else 0
    d.num_decode_tokens = T - d.num_prefill_tokens
    for f, k in (("token_ids", "token_ids"), ("positions", "positions"), ("cu_q", "cu_q"), ("kv_len", "kv_len"),
                 ("block_table", "block_table"), ("sample_token_idx", "sample_idx")):
        setattr(d, f, _p32(keep[k]))
    if "slot_mapping" in keep:
        d.slot_mapping = _p32(keep["slot_mapping"])
    if "seq_req_ids" in keep:
        d.seq_req_ids = keep["seq_req_ids"].ctypes.data_as(_P64)
    return d, keep


class Stage:
    """Owner of a gllm_stage*: weights [layer_begin, layer_end), paged KV cache, workspaces."""

    def __init__(self, m, layer_begin, layer_end, kv_blocks, max_tokens, max_seqs, device=0, block_size=16):
        self.m = m
        self.cfg = model_cfg(m)
        self.layer_begin, self.layer_end = layer_begin, layer_end
        self.max_tokens, self.max_seqs = max_tokens, max_seqs
        h = C.c_void_p()
        _check(lib().gllm_init_stage(C.byref(self.cfg), layer_begin, layer_end, kv_blocks, block_size,
                                     max_tokens, max_seqs, device, C.byref(h)))
        self.h = h

    def close(self):
        if getattr(self, "h", None) and _lib is not None:
            _lib.gllm_free_stage(self.h)
            self.h = None

    __del__ = close

    def forward(self, desc: BatchDesc, hidden_in=0, hidden_out=0, sampled_out=0, stream=0):
        """Enqueue stage_forward; buffers are raw device pointers (ints), stream a cudaStream_t int."""
        return _check(lib().gllm_stage_forward(self.h, C.byref(desc), hidden_in or None, hidden_out or None,
                                               sampled_out or None, stream or None))

    def prepare(self, desc: BatchDesc, stream=0) -> int:
        """Phase 1 (metadata): validate + copy the batch metadata to the device; returns a handle."""
        h = C.c_int32()
        _check(lib().gllm_stage_prepare(self.h, C.byref(desc), stream or None, C.byref(h)))
        return h.value

    def forward_prepared(self, handle, hidden_in=0, hidden_out=0, sampled_out=0, stream=0):
        """Phase 2 (activations): launch the layers of a prepared batch."""
        return _check(lib().gllm_stage_forward_prepared(self.h, handle, hidden_in or None, hidden_out or None,
                                                        sampled_out or None, stream or None))

    def release(self, handle):
        _check(lib().gllm_stage_release(self.h, handle))

    def sync(self):
        _check(lib().gllm_stage_sync(self.h))

    def set_deterministic(self, on=True):
        _check(lib().gllm_stage_set_deterministic(self.h, int(on)))

    def set_profiling(self, on=True):
        _check(lib().gllm_stage_set_profiling(self.h, int(on)))

    def last_timing(self) -> dict:
        out = (C.c_float * len(TIMING_NAMES))()
        _check(lib().gllm_stage_last_timing(self.h, out, len(TIMING_NAMES)))
        return dict(zip(TIMING_NAMES, list(out)))

    def last_launches(self) -> int:
        n = C.c_int32()
        _check(lib().gllm_stage_last_launches(self.h, C.byref(n)))
        return n.value

    def read_weight(self, layer, name, row0, nrows, cols):
        out = np.zeros((nrows, cols), np.float32)
        _check(lib().gllm_stage_read_weight(self.h, layer, name.encode(), row0, nrows,
                                            out.ctypes.data_as(C.POINTER(C.c_float))))
        return out

    def read_kv(self, layer, slots):
        slots = np.ascontiguousarray(slots, dtype=np.int32)
        n = slots.shape[0]
        k = np.zeros((n, self.m.n_kv_heads, self.m.head_dim), np.float32)
        v = np.zeros_like(k)
        _check(lib().gllm_stage_read_kv(self.h, layer, _p32(slots), n, k.ctypes.data_as(C.POINTER(C.c_float)),
                                        v.ctypes.data_as(C.POINTER(C.c_float))))
        return k, v

    def read_slots(self, n):
        out = np.zeros(n, np.int32)
        _check(lib().gllm_stage_read_slots(self.h, _p32(out), n))
        return out

    def fill_warm_kv(self, req_ids, context_lens, block_table):
        """gllm_stage_fill_warm_kv: block_table int32 [n, max_blocks] (rows -1 padded)."""
        rid = np.ascontiguousarray(req_ids, dtype=np.int64)
        ctx = np.ascontiguousarray(context_lens, dtype=np.int32)
        bt = np.ascontiguousarray(block_table, dtype=np.int32)
        n = int(rid.shape[0])
        mb = int(bt.shape[1]) if bt.ndim == 2 else 0
        _check(lib().gllm_stage_fill_warm_kv(self.h, n, rid.ctypes.data_as(C.POINTER(C.c_int64)), _p32(ctx),
                                             _p32(bt), mb))

    # pipeline hand-off (NCCL P2P)
    def comm_init(self, unique_id: bytes, rank: int, world: int):
        buf = C.create_string_buffer(unique_id, 128)
        _check(lib().gllm_comm_init(self.h, buf, rank, world))

    # fused peer hand-off (a12): see include/gllm.h gllm_peer_*
    def peer_ring_create(self, depth: int) -> bytes:
        buf = C.create_string_buffer(128)
        _check(lib().gllm_peer_ring_create(self.h, depth, buf))
        return buf.raw

    def peer_ring_open(self, handle: bytes) -> bytes:
        """Maps the receiver's ring; returns the handle of this sender's slot credits."""
        buf = C.create_string_buffer(handle, 128)
        out = C.create_string_buffer(128)
        _check(lib().gllm_peer_ring_open(self.h, buf, out))
        return out.raw

    def peer_credit_open(self, credit_handle: bytes):
        buf = C.create_string_buffer(credit_handle, 128)
        _check(lib().gllm_peer_credit_open(self.h, buf))

    def forward_prepared_peer(self, handle, tick, hidden_in=0, stream=0):
        return _check(lib().gllm_stage_forward_prepared_peer(self.h, handle, hidden_in or None, tick, stream or None))

    def peer_ring_recv(self, tick, stream=0) -> int:
        out = C.c_void_p()
        _check(lib().gllm_peer_ring_recv(self.h, tick, stream or None, C.byref(out)))
        return out.value

    def comm_size(self):
        """(nranks, rank) of this stage's NCCL communicator."""
        n, r = C.c_int32(), C.c_int32()
        _check(lib().gllm_comm_size(self.h, C.byref(n), C.byref(r)))
        return n.value, r.value

    def send_hidden(self, ptr, num_tokens, dst, stream=0):
        _check(lib().gllm_send_hidden(self.h, ptr, num_tokens, dst, stream or None))

    def recv_hidden(self, ptr, num_tokens, src, stream=0):
        _check(lib().gllm_recv_hidden(self.h, ptr, num_tokens, src, stream or None))


def op_gemm(A_ptr, W_ptr, M, N, K, epi, out_ptr, bias_ptr=0, stream=0):
    """gllm_op_gemm (include/gllm_ops.h): the stage's tcgen05 GEMM on raw device pointers."""
    _check(lib().gllm_op_gemm(A_ptr, W_ptr, M, N, K, epi, bias_ptr or None, out_ptr, stream or None))


def op_set_deterministic(on: bool):
    _check(lib().gllm_op_set_deterministic(int(on)))


def op_set_gemm_variant(cta_group: int):
    """0 = automatic, 1 = 1-CTA 128x256 kernel, 2 = CTA-pair 256x256 kernel (testing / tuning)."""
    _check(lib().gllm_op_set_gemm_variant(cta_group))


def get_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _check(lib().gllm_get_unique_id(buf))
    return buf.raw


def init_stage(m, layer_begin, layer_end, kv_blocks, max_tokens, max_seqs, device=0) -> Stage:
    return Stage(m, layer_begin, layer_end, kv_blocks, max_tokens, max_seqs, device)
