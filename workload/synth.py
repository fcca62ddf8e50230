"""Seeded synthetic inputs shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the method: it only draws random numbers
and integer layouts (lengths, block tables) with the shapes of the paper's
workloads (DESIGN.md §6 "Input recipe").  Both sides — ``oracle`` and the
product ``paper_conf_asplos_0001xc0l026_b200`` — read the same tensors from
here; neither side imports the other.

Seeds (fixed): weights 0, activations 1, block tables 2, lengths 3.

Model shapes are the public HF configs of the architectures the paper and
BASELINE.json name (Llama-3.1-8B; Qwen2.5-14B and Llama-3.1-70B from
BASELINE.json configs 4-5).  Weights are random-init: N(0, 1/fan_in), RMSNorm
gains 1 + 0.05 N(0,1), Qwen QKV bias 0.02 N(0,1).
"""
from __future__ import annotations

from dataclasses import dataclass, field, asdict

import numpy as np
import torch

SEED_WEIGHTS, SEED_ACT, SEED_TABLES, SEED_LENGTHS = 0, 1, 2, 3


@dataclass
class ModelShape:
    name: str
    d_model: int
    n_heads: int
    n_kv_heads: int
    head_dim: int
    d_ff: int
    n_layers: int
    dtype: str = "bf16"            # "bf16" or "fp32"
    rms_eps: float = 1e-5
    rope_theta: float = 500000.0
    rope_llama3: int = 1
    rope_factor: float = 8.0
    rope_low_freq: float = 1.0
    rope_high_freq: float = 4.0
    rope_orig_max_pos: int = 8192
    qkv_bias: int = 0

    @property
    def n_qkv(self) -> int:
        return (self.n_heads + 2 * self.n_kv_heads) * self.head_dim

    def shard(self, tp: int) -> "ModelShape":
        """Per-rank shape under Megatron tensor parallelism (heads / FFN split)."""
        assert self.n_heads % tp == 0 and self.n_kv_heads % tp == 0 and self.d_ff % tp == 0
        s = ModelShape(**asdict(self))
        s.n_heads //= tp; s.n_kv_heads //= tp; s.d_ff //= tp
        return s


MODELS = {
    # BASELINE.json config 1 (DESIGN R-6: Hkv = 2, hd = 64, I = 768)
    "tiny": ModelShape("tiny", 256, 4, 2, 64, 768, 2, dtype="fp32", rope_theta=10000.0,
                       rope_llama3=0),
    "llama3.1-8b": ModelShape("llama3.1-8b", 4096, 32, 8, 128, 14336, 32),
    "qwen2.5-14b": ModelShape("qwen2.5-14b", 5120, 40, 8, 128, 13824, 48, rope_theta=1e6,
                              rope_llama3=0, qkv_bias=1),
    "llama3.1-70b": ModelShape("llama3.1-70b", 8192, 64, 8, 128, 28672, 80),
}


@dataclass
class Workload:
    """One co-run step's request mix (BASELINE.json configs)."""
    name: str
    model: str
    prefill_lens: list                 # new tokens per prefill request (ctx 0)
    decode_ctx: list                   # cached tokens per decode request (1 new each)
    block_size: int = 16
    tp: int = 1
    extra: dict = field(default_factory=dict)


def _sharegpt_lens(rng, n, total):
    """ShareGPT-shaped prompt lengths: lognormal(ln 400, 0.8) clipped to
    [32, 2048], rescaled so they sum to ``total`` (SURVEY §8d recipe)."""
    x = np.clip(rng.lognormal(np.log(400.0), 0.8, size=n), 32, 2048)
    x = np.maximum(1, np.floor(x * total / x.sum())).astype(np.int64)
    x[np.argmax(x)] += total - x.sum()
    return [int(v) for v in x]


def workload(name: str) -> Workload:
    rng = np.random.default_rng(SEED_LENGTHS)
    if name == "tiny":          # config 1
        return Workload(name, "tiny", [128], [64] * 4)
    if name == "sharegpt-8b":   # config 2
        return Workload(name, "llama3.1-8b", _sharegpt_lens(rng, 8, 4096),
                        [int(v) for v in rng.integers(512, 1537, size=128)])
    if name == "arxiv-8b":      # config 3
        return Workload(name, "llama3.1-8b", [8192],
                        [int(v) for v in rng.integers(2048, 6145, size=256)])
    if name.startswith("qwen14b-tp"):   # config 4 (tp 2 or 4)
        tp = int(name[len("qwen14b-tp"):])
        pre = _sharegpt_lens(rng, 8, 4096) + [8192]
        dec = [int(v) for v in rng.integers(512, 1537, size=128)] + \
              [int(v) for v in rng.integers(2048, 6145, size=64)]
        return Workload(name, "qwen2.5-14b", pre, dec, tp=tp)
    if name == "llama70b-tp8":  # config 5
        return Workload(name, "llama3.1-70b", [8192, 8192],
                        [int(v) for v in rng.integers(2048, 6145, size=512)], tp=8)
    raise KeyError(name)


def small_workload(model: str, prefill_lens, decode_ctx, block_size=16) -> Workload:
    return Workload("custom", model, list(prefill_lens), list(decode_ctx), block_size)


# --------------------------------------------------------------------- tensors

def _gen(seed: int, device="cpu") -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    return g


def _store(t: torch.Tensor, dtype: str) -> torch.Tensor:
    """Values as the model stores them (bf16-exact float32 for bf16 models)."""
    return t.bfloat16().float() if dtype == "bf16" else t.float()


def layer_weights(m: ModelShape, layer: int, device="cpu") -> dict:
    """Random-init weights of one layer, float32 tensors holding the stored
    values.  Layout (all row-major, nn.Linear [out][in]):
      w_qkv [(H+2Hkv)hd][d] (q heads, k heads, v heads), b_qkv [(H+2Hkv)hd] | None,
      w_o [d][H hd], w_gate_up [2I][d] (gate rows then up rows), w_down [d][I],
      g_attn [d], g_mlp [d]."""
    g = _gen(SEED_WEIGHTS * 1_000_003 + 7919 * layer + 1, device)
    d, I, nq = m.d_model, m.d_ff, m.n_qkv

    def rn(*shape, std):
        return torch.randn(*shape, generator=g, device=device) * std
    w = {
        "w_qkv": _store(rn(nq, d, std=d ** -0.5), m.dtype),
        "b_qkv": _store(rn(nq, std=0.02), m.dtype) if m.qkv_bias else None,
        "w_o": _store(rn(d, m.n_heads * m.head_dim, std=(m.n_heads * m.head_dim) ** -0.5), m.dtype),
        "w_gate_up": _store(rn(2 * I, d, std=d ** -0.5), m.dtype),
        "w_down": _store(rn(d, I, std=I ** -0.5), m.dtype),
        "g_attn": _store(1.0 + 0.05 * rn(d, std=1.0), m.dtype),
        "g_mlp": _store(1.0 + 0.05 * rn(d, std=1.0), m.dtype),
    }
    return w


def shard_weights(m: ModelShape, w: dict, tp: int, rank: int) -> dict:
    """Megatron split of one layer's weights for rank ``rank`` of ``tp``:
    QKV and gate/up column-parallel by heads / FFN rows, O-proj and down
    row-parallel (input columns).  Pure slicing — no arithmetic."""
    H, Hkv, hd, I = m.n_heads, m.n_kv_heads, m.head_dim, m.d_ff
    h0, h1 = rank * H // tp, (rank + 1) * H // tp
    g0, g1 = rank * Hkv // tp, (rank + 1) * Hkv // tp
    i0, i1 = rank * I // tp, (rank + 1) * I // tp
    rows = list(range(h0 * hd, h1 * hd)) + \
        list(range((H + g0) * hd, (H + g1) * hd)) + \
        list(range((H + Hkv + g0) * hd, (H + Hkv + g1) * hd))
    rows = torch.tensor(rows, device=w["w_qkv"].device)
    out = {
        "w_qkv": w["w_qkv"][rows].contiguous(),
        "b_qkv": None if w["b_qkv"] is None else w["b_qkv"][rows].contiguous(),
        "w_o": w["w_o"][:, h0 * hd:h1 * hd].contiguous(),
        "w_gate_up": torch.cat([w["w_gate_up"][i0:i1], w["w_gate_up"][I + i0:I + i1]]).contiguous(),
        "w_down": w["w_down"][:, i0:i1].contiguous(),
        "g_attn": w["g_attn"], "g_mlp": w["g_mlp"],
    }
    return out


def hidden(n: int, d: int, seed_offset=0, device="cpu") -> torch.Tensor:
    """Residual-stream input x ~ N(0,1), fp32."""
    return torch.randn(n, d, generator=_gen(SEED_ACT * 1_000_003 + 17 + seed_offset, device),
                       device=device)


@dataclass
class PagedLayout:
    n_blocks: int
    block_size: int
    max_blocks: int
    block_table: np.ndarray      # int32 [n_reqs][max_blocks], -1 padded... filled with valid ids
    q_lens: np.ndarray           # int32 [n_reqs]
    ctx_lens: np.ndarray         # int32 [n_reqs]


def paged_layout(q_lens, ctx_lens, block_size=16, slack=0.25, seed_offset=0,
                 min_blocks=0) -> PagedLayout:
    """Block tables for a batch: each request needs ceil((ctx+q)/B) blocks;
    the pool has 25% slack blocks; ids come from a random permutation of the
    free list (fragmented).  Unused table entries hold 0 (never read)."""
    rng = np.random.default_rng(SEED_TABLES * 1_000_003 + seed_offset)
    q_lens = np.asarray(q_lens, dtype=np.int32)
    ctx_lens = np.asarray(ctx_lens, dtype=np.int32)
    need = [(-(-int(c + q) // block_size)) for c, q in zip(ctx_lens, q_lens)]
    total = int(sum(need))
    n_blocks = max(min_blocks, int(np.ceil(total * (1.0 + slack))) + 1)
    perm = rng.permutation(n_blocks).astype(np.int32)
    max_blocks = max(1, max(need) if need else 1)
    bt = np.zeros((len(need), max_blocks), dtype=np.int32)
    pos = 0
    for r, nb in enumerate(need):
        bt[r, :nb] = perm[pos:pos + nb]
        pos += nb
    return PagedLayout(n_blocks, block_size, max_blocks, bt, q_lens, ctx_lens)


def kv_pool(m: ModelShape, n_blocks: int, block_size: int, layer: int, device="cpu"):
    """KV pool [n_blocks][Hkv][B][hd] pre-filled with N(0,1) values (the cached
    context "as if produced by an earlier prefill"), stored dtype values."""
    g = _gen(SEED_ACT * 1_000_003 + 104729 * (layer + 1), device)
    shape = (n_blocks, m.n_kv_heads, block_size, m.head_dim)
    k = _store(torch.randn(*shape, generator=g, device=device), m.dtype)
    v = _store(torch.randn(*shape, generator=g, device=device), m.dtype)
    return k, v


def combined_batch(wl: Workload):
    """Prefill requests first, then decode requests, in one block-table space
    (disjoint block sets).  Returns (q_lens, ctx_lens, n_prefill_reqs)."""
    q = list(wl.prefill_lens) + [1] * len(wl.decode_ctx)
    c = [0] * len(wl.prefill_lens) + list(wl.decode_ctx)
    return q, c, len(wl.prefill_lens)
