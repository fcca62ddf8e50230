"""Tensor-parallel host logic on CPU (world size 2, gloo): the product's
sharding (parallel.py) composed the way bullet_step composes it (per-rank
attention on local heads, fp32 partial sums all-reduced after O-proj and
down) reproduces the unsharded oracle layer; the NCCL id exchange gives every
rank the same bytes.  Oracle primitives compute each rank's arithmetic."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle as O
from paper_conf_asplos_0001xc0l026_b200 import parallel
from paper_conf_asplos_0001xc0l026_b200.bullet import Model
from workload import synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


M = synth.ModelShape("tp-test", 64, 4, 2, 16, 96, 1, dtype="bf16", rope_theta=10000.0, rope_llama3=0,
                     qkv_bias=1)


def _cfg(m):
    return O.OracleCfg(d_model=m.d_model, n_heads=m.n_heads, n_kv_heads=m.n_kv_heads, head_dim=m.head_dim,
                       d_ff=m.d_ff, rms_eps=m.rms_eps, rope_theta=m.rope_theta, rope_llama3=0, bf16_mirror=1)


def _rank_partials(rank, tp, q_lens, ctx, lay, x, w, pk, pv):
    """One rank's S1-S9 with an all-reduce after S5 and S8 (oracle arithmetic)."""
    model = Model.of(M)
    ws = parallel.shard_layer_weights({k: (None if v is None else torch.from_numpy(v)) for k, v in w.items()},
                                      model, tp, rank)
    ws = {k: (None if v is None else v.numpy()) for k, v in ws.items()}
    lm = parallel.shard_model(model, tp)
    cfg = _cfg(M)
    cfg_l = O.OracleCfg(**{**cfg.__dict__, "n_heads": lm.n_heads, "n_kv_heads": lm.n_kv_heads, "d_ff": lm.d_ff})
    pk_l = parallel.shard_kv_pool(torch.from_numpy(pk), tp, rank).numpy().copy()
    pv_l = parallel.shard_kv_pool(torch.from_numpy(pv), tp, rank).numpy().copy()
    # attention half of the layer with W_o, W_down zero -> out = x exactly; the
    # local o comes from the oracle diagnostics
    zero = dict(ws, w_o=np.zeros_like(ws["w_o"]), w_down=np.zeros_like(ws["w_down"]))
    _, dg = O.layer_forward(cfg_l, zero, pk_l, pv_l, q_lens, ctx, lay.block_table, x, diag=True)
    part_o = O.linear(dg["o"], ws["w_o"])                                     # row-parallel O-proj
    t = torch.from_numpy(part_o)
    dist.all_reduce(t)                                                        # S9 (fp32/fp64 sum)
    x1 = x + t.numpy()
    h2 = O.round_bf16(O.rmsnorm(x1, ws["g_mlp"], cfg.rms_eps))
    gu = O.linear(h2, ws["w_gate_up"])
    Il = lm.d_ff
    a = O.round_bf16(gu[:, :Il] / (1 + np.exp(-gu[:, :Il])) * gu[:, Il:])
    t = torch.from_numpy(O.linear(a, ws["w_down"]))
    dist.all_reduce(t)
    return x1 + t.numpy()


def _worker(rank, tp, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=tp)
    try:
        rng = np.random.default_rng(0)
        q_lens, ctx = [9, 1, 1], [0, 20, 33]
        lay = synth.paged_layout(q_lens, ctx, 16)
        w = {k: (None if v is None else v.numpy()) for k, v in synth.layer_weights(M, 0).items()}
        pk, pv = synth.kv_pool(M, lay.n_blocks, 16, 0)
        pk, pv = pk.numpy(), pv.numpy()
        x = rng.standard_normal((sum(q_lens), M.d_model))
        out_tp = _rank_partials(rank, tp, q_lens, ctx, lay, x, w, pk, pv)
        ref = O.layer_forward(_cfg(M), w, pk.copy(), pv.copy(), q_lens, ctx, lay.block_table, x)
        uids = parallel.nccl_uids(make=lambda: bytes([7]) * 128)
        # PEER mode bootstrap: every rank's 64-byte IPC handle, in rank order
        handles = parallel.gather_bytes(bytes([rank + 1]) * 64)
        q.put((rank, float(np.abs(out_tp - ref).max()), len(uids), uids[:4], handles))
    finally:
        dist.destroy_process_group()


def test_tp2_sharded_layer_equals_unsharded_oracle():
    tp = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, tp, port, q)) for r in range(tp)]
    for p in ps:
        p.start()
    res = [q.get(timeout=240) for _ in range(tp)]
    for p in ps:
        p.join(60)
        assert p.exitcode == 0
    for rank, err, n, head, handles in res:
        assert err < 1e-9, (rank, err)      # same bf16 rounding points, fp64 sums
        assert n == 256 and head == bytes([7]) * 4
        assert handles == b"".join(bytes([r + 1]) * 64 for r in range(tp))


def test_shard_shapes_all_tp_configs():
    for name, tp in (("qwen2.5-14b", 2), ("qwen2.5-14b", 4), ("llama3.1-70b", 8)):
        m = Model.of(synth.MODELS[name])
        lm = parallel.shard_model(m, tp)
        assert lm.n_heads * tp == m.n_heads and lm.n_kv_heads * tp == m.n_kv_heads
        # every GEMM dimension of the shard stays tileable by the tcgen05 kernels
        nq = (lm.n_heads + 2 * lm.n_kv_heads) * lm.head_dim
        assert nq % 64 == 0 and lm.d_ff % 64 == 0 and (lm.n_heads * lm.head_dim) % 64 == 0
    with pytest.raises(ValueError):
        parallel.shard_model(Model.of(synth.MODELS["llama3.1-70b"]), 16)
