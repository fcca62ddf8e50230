"""Tensor parallelism through the NCCL all-reduce (bullet_create with
ncclUniqueIds: the non-lead ranks write their fp32 partials into the
residual stream and an in-place ncclAllReduce(float32) after O-proj and
after down restores x + sum of partials, one communicator per phase).
Needs one GPU per rank (NCCL refuses two ranks on one device): runs on a
box with >= 2 GPUs, skips on one.  Two processes, TP2, two layers: every
rank's hidden equal, and each layer step within the north-star bar of the
unsharded oracle layer fed the same input."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

PRE_LENS, DEC_CTX = [200, 33], [64, 1, 300, 17]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank(rank, tp, port, q):
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    sys.path[:0] = [here, os.path.dirname(here)]
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch
    import torch.distributed as dist
    from harness import Setup, compare, oracle_layer
    from workload import synth
    import paper_conf_asplos_0001xc0l026_b200 as B
    from paper_conf_asplos_0001xc0l026_b200 import parallel
    torch.cuda.set_device(rank)
    dist.init_process_group("gloo", rank=rank, world_size=tp)
    try:
        M = synth.ModelShape("tp-nccl", 1024, 8, 4, 128, 2048, 2)
        S = Setup(M, PRE_LENS, DEC_CTX, n_layers=2)
        S.bl.close()
        lm = parallel.shard_model(B.Model.of(M), tp)
        pools = [(parallel.shard_kv_pool(k, tp, rank), parallel.shard_kv_pool(v, tp, rank)) for k, v in S.pool_gpu]
        bl = B.Bullet(lm, pools, max_prefill_tokens=sum(PRE_LENS), max_decode_tokens=len(DEC_CTX),
                      max_position=2048, tp_size=tp, tp_rank=rank, nccl_uids=parallel.nccl_uids())
        for l in range(2):
            bl.set_layer_weights(l, parallel.shard_layer_weights(S.w_gpu[l], B.Model.of(M), tp, rank))
        bt = S.lay.block_table
        x_pre, x_dec = S.x_pre.cuda(), S.x_dec.cuda()
        errs = []
        for l in range(2):   # per layer step (R-4c), NCCL all-reduce after O-proj and down
            pre = B.Batch(PRE_LENS, [0] * len(PRE_LENS), bt[:S.n_pre], x_pre.clone(), l, l + 1)
            dec = B.Batch([1] * len(DEC_CTX), DEC_CTX, bt[S.n_pre:], x_dec.clone(), l, l + 1)
            torch.cuda.synchronize()
            bl.step(pre, dec, 74, B.CORUN)
            bl.sync()
            ref = oracle_layer(S, l, x_pre.cpu().numpy(), x_dec.cpu().numpy())
            for name, b in (("pre", pre), ("dec", dec)):
                errs.append(compare(b.hidden.cpu().numpy(), ref[name]))
            x_pre, x_dec = pre.hidden, dec.hidden
        digest = float(x_pre.double().sum() + x_dec.double().sum())
        q.put((rank, errs, digest))
        bl.close()
    finally:
        dist.destroy_process_group()


def test_nccl_tp2_two_layers_match_oracle():
    if torch.cuda.device_count() < 2:
        pytest.skip("NCCL tensor parallelism needs one GPU per rank (this box has %d)" % torch.cuda.device_count())
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_rank, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=600) for _ in ps]
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    out.sort()
    assert out[0][2] == out[1][2]                      # every rank holds the same residual stream
    for rank, errs, _ in out:
        for mx, mr in errs:
            assert mx <= 2e-2 and mr <= 1e-3, (rank, mx, mr)
