"""Tensor parallelism for the larger models (BASELINE configs 4-5; north_star
(4)): Megatron column/row sharding of one layer and the NCCL bootstrap.

QKV and gate/up are column-parallel (rank r owns query heads
[r H/tp, (r+1) H/tp), kv heads [r Hkv/tp, ...) and FFN rows [r I/tp, ...));
O-proj and down are row-parallel (the matching input columns).  Inside
`bullet_step` the non-lead ranks write their fp32 partial products into the
residual stream and an in-place ncclAllReduce(float32, sum) after S5 and S8
restores x + sum of partials.  In PEER mode (no ncclUniqueIds)
the O-proj / down GEMMs reduce over the ranks' symmetric buffers themselves
(fused, smid-gated); `connect_peers` exchanges the
cudaIpcMemHandles.  KV pools shard by kv head; block tables are replicated.
torch.distributed is used only to launch ranks and to exchange these few
bytes."""
from __future__ import annotations

import torch

from .bullet import Model, nccl_unique_id


def shard_model(model: Model, tp: int) -> Model:
    """Per-rank model shape (local heads / FFN width; d_model unchanged)."""
    if model.n_heads % tp or model.n_kv_heads % tp or model.d_ff % tp:
        raise ValueError(f"heads {model.n_heads}/{model.n_kv_heads} and d_ff {model.d_ff} must divide tp={tp}")
    kw = {k: getattr(model, k) for k in Model.__dataclass_fields__}
    kw.update(n_heads=model.n_heads // tp, n_kv_heads=model.n_kv_heads // tp, d_ff=model.d_ff // tp)
    return Model(**kw)


def shard_layer_weights(w: dict, model: Model, tp: int, rank: int) -> dict:
    """Rank `rank`'s slice of one layer's full weights (dict of tensors in the
    bullet_layer_weights layout).  Returns contiguous tensors on w's device."""
    H, Hkv, hd, I = model.n_heads, model.n_kv_heads, model.head_dim, model.d_ff
    h0, h1 = rank * H // tp, (rank + 1) * H // tp
    g0, g1 = rank * Hkv // tp, (rank + 1) * Hkv // tp
    i0, i1 = rank * I // tp, (rank + 1) * I // tp
    dev = w["w_qkv"].device
    rows = torch.cat([torch.arange(h0 * hd, h1 * hd), torch.arange((H + g0) * hd, (H + g1) * hd),
                      torch.arange((H + Hkv + g0) * hd, (H + Hkv + g1) * hd)]).to(dev)
    return {
        "w_qkv": w["w_qkv"].index_select(0, rows).contiguous(),
        "b_qkv": None if w.get("b_qkv") is None else w["b_qkv"].index_select(0, rows).contiguous(),
        "w_o": w["w_o"][:, h0 * hd:h1 * hd].contiguous(),
        "w_gate_up": torch.cat([w["w_gate_up"][i0:i1], w["w_gate_up"][I + i0:I + i1]]).contiguous(),
        "w_down": w["w_down"][:, i0:i1].contiguous(),
        "g_attn": w["g_attn"].contiguous(), "g_mlp": w["g_mlp"].contiguous(),
    }


def shard_kv_pool(pool: torch.Tensor, tp: int, rank: int) -> torch.Tensor:
    """[n_blocks][Hkv][B][hd] -> this rank's kv heads."""
    Hkv = pool.shape[1]
    return pool[:, rank * Hkv // tp:(rank + 1) * Hkv // tp].contiguous()


def nccl_uids(group=None, make=nccl_unique_id) -> bytes:
    """Two ncclUniqueIds (prefill and decode communicators), created on rank 0
    and broadcast to every rank of `group` (256 bytes, identical everywhere)."""
    import torch.distributed as dist
    rank = dist.get_rank(group)
    obj = [make() + make() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group else 0, group=group)
    return obj[0]


def gather_bytes(blob: bytes, group=None) -> bytes:
    """Every rank's `blob` (equal lengths), concatenated in rank order."""
    import torch.distributed as dist
    out = [None] * dist.get_world_size(group)
    dist.all_gather_object(out, blob, group=group)
    if len({len(b) for b in out}) != 1:
        raise ValueError("ranks sent blobs of different lengths")
    return b"".join(out)


def connect_peers(bl, group=None):
    """PEER mode, one process per GPU: exchange the symmetric regions'
    cudaIpcMemHandles and connect (bullet_tp_connect_ipc)."""
    bl.tp_connect_ipc(gather_bytes(bl.tp_ipc_handle(), group))
