"""Model shapes, scheduler hyper-parameters and stream recipes (data only).

Sources (PAPER.md = /root/reference/PAPER.md):
  * model families: Qwen2.5-14B/32B, Llama-3.1 ("100B") -- PAPER.md L218, L224;
    exact dimensions are the public HF configs ([ext]).
  * Token-Throttling defaults #T=8, #MaxP=2048, #MinP=32, KV_thresh=0.05 -- L248;
    max sequences 1024 -- L575; KV block of 16 tokens -- BASELINE.json configs.
"""
from __future__ import annotations

from dataclasses import dataclass, replace


@dataclass(frozen=True)
class ModelShape:
    name: str
    n_layers: int
    hidden: int
    n_heads: int
    n_kv_heads: int
    head_dim: int
    intermediate: int
    vocab: int
    rms_eps: float
    rope_theta: float
    qkv_bias: bool
    weight_seed: int

    @property
    def q_dim(self) -> int:
        return self.n_heads * self.head_dim

    @property
    def kv_dim(self) -> int:
        return self.n_kv_heads * self.head_dim

    def with_layers(self, n: int) -> "ModelShape":
        return replace(self, n_layers=n)


@dataclass(frozen=True)
class SchedParams:
    """Mirror of `gllm_sched_cfg` (include/gllm.h)."""
    iterp: int = 8            # #T   (L151, L248)
    maxp: int = 2048          # #MaxP (L151, L248)
    minp: int = 32            # #MinP (L151, L248)
    kvthresh_num: int = 1     # KV_thresh = num/den = 0.05 (L165, L248)
    kvthresh_den: int = 20
    pp_depth: int = 1         # #PP_depth (L181)
    num_blocks: int = 64
    block_size: int = 16
    max_seqs: int = 1024      # L575
    policy: int = 0           # 0 = Token Throttling; 1 = Sarathi-Serve; 2 = w/o WT; 3 = w/o UT (§4.5); 4 = R21
    token_budget: int = 2048  # Sarathi only (L248)
    attn_pairs_per_token: int = 0  # policy 4 (context-aware throttling, R21, L354) only

    def with_(self, **kw) -> "SchedParams":
        return replace(self, **kw)


# weight seeds: 1000 + config index
MODELS = {
    # C0: BASELINE.json gives hidden 256 / 4 heads / 16-token blocks; I, V, theta are ours (SURVEY §8c note 2)
    "C0": ModelShape("tiny", 2, 256, 4, 4, 64, 1024, 512, 1e-5, 10000.0, False, 1000),
    "C1": ModelShape("llama3-8b", 32, 4096, 32, 8, 128, 14336, 128256, 1e-5, 500000.0, False, 1001),
    "C2": ModelShape("qwen2.5-14b", 48, 5120, 40, 8, 128, 13824, 152064, 1e-5, 1e6, True, 1002),
    "C3": ModelShape("qwen2.5-32b", 64, 5120, 40, 8, 128, 27648, 152064, 1e-5, 1e6, True, 1003),
    "C4": ModelShape("llama3-70b", 80, 8192, 64, 8, 128, 28672, 128256, 1e-5, 500000.0, False, 1004),
}

SCHED = {
    "C0": SchedParams(iterp=1, pp_depth=1, num_blocks=64),
    "C0b": SchedParams(iterp=1, maxp=40, pp_depth=1, num_blocks=64),
    "C1": SchedParams(pp_depth=2, num_blocks=100000),
    "C2": SchedParams(pp_depth=4, num_blocks=36864),
    "C3": SchedParams(pp_depth=8, num_blocks=65536),
    "C4": SchedParams(pp_depth=8, num_blocks=154624),
}

# Stream recipes (SURVEY.md §8(d) "Synthetic streams").
STREAMS = {
    "C0": dict(kind="handmade_c0"),
    "C0b": dict(kind="handmade_c0b"),
    "C1": dict(kind="lognormal", seed=1, n=12000, rate=6.0,
               prompt=(180.0, 0.9, 4, 4096), output=(140.0, 0.8, 2, 1024), window=(400, None)),
    "C2": dict(kind="lognormal", seed=2, n=12000, rate=6.0,
               prompt=(180.0, 0.9, 4, 4096), output=(140.0, 0.8, 2, 1024), window=(800, None)),
    "C3": dict(kind="lognormal", seed=3, n=600, rate=0.5,
               prompt=(4096.0, 0.5, 1024, 32768), output=(128.0, 0.7, 2, 1024), window=(400, 1100)),
    "C4": dict(kind="lognormal", seed=4, n=6000, rate=1.0,
               prompt=(1024.0, 0.5, 128, 4096), output=(768.0, 0.5, 128, 2048), window=(400, 3000),
               warm=dict(n=1024, context=(1536, 2560), remaining=(256, 1024))),
}


def config(name: str):
    """(ModelShape, SchedParams, stream recipe) for a config name C0..C4 / C0b."""
    model = MODELS["C0" if name == "C0b" else name]
    return model, SCHED[name], STREAMS[name]
