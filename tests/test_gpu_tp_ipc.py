"""Fused all-reduce (PEER mode) through the real multi-process path: two
processes, one rank each, both on the one B200 of the test box.  Each rank
exports its symmetric region with bullet_tp_ipc_handle, the handles are
exchanged over torch.distributed (gloo), every rank opens the other's with
bullet_tp_connect_ipc (cudaIpcOpenMemHandle) and steps its shard.  Two CUDA
contexts share the GPU by time slices (no MPS), so the ranks' kernels wait
on each other across context switches — slower than ranks on two GPUs, but
the same code path, cross-process memory ordering included.  Checked: both
ranks hold bit-identical residual streams that match the unsharded oracle
layer."""
import os
import socket

import numpy as np
import pytest
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
    from harness import Setup
    from workload import synth
    import paper_conf_asplos_0001xc0l026_b200 as B
    from paper_conf_asplos_0001xc0l026_b200 import parallel
    dist.init_process_group("gloo", rank=rank, world_size=tp)
    try:
        torch.cuda.set_device(0)
        M = synth.ModelShape("tp-ipc", 1024, 8, 4, 128, 2048, 1)
        S = Setup(M, PRE_LENS, DEC_CTX, n_layers=1)
        S.bl.close()
        lm = parallel.shard_model(B.Model.of(M), tp)
        pools = [(parallel.shard_kv_pool(k, tp, rank), parallel.shard_kv_pool(v, tp, rank)) for k, v in S.pool_gpu]
        bl = B.Bullet(lm, pools, max_prefill_tokens=sum(PRE_LENS), max_decode_tokens=len(DEC_CTX),
                      max_position=2048, tp_size=tp, tp_rank=rank)
        bl.set_layer_weights(0, parallel.shard_layer_weights(S.w_gpu[0], B.Model.of(M), tp, rank))
        parallel.connect_peers(bl)                    # IPC handles over gloo -> cudaIpcOpenMemHandle
        bt = S.lay.block_table
        hp = bl.tp_hidden(0, S.x_pre.shape[0]); hp.copy_(S.x_pre.cuda())
        hd = bl.tp_hidden(1, S.x_dec.shape[0]); hd.copy_(S.x_dec.cuda())
        pre = B.Batch(PRE_LENS, [0] * len(PRE_LENS), bt[:S.n_pre], hp, 0, 1)
        dec = B.Batch([1] * len(DEC_CTX), DEC_CTX, bt[S.n_pre:], hd, 0, 1)
        torch.cuda.synchronize()
        dist.barrier()
        g = 36
        sp, sd = torch.cuda.Stream(), torch.cuda.Stream()
        bl.step_ranges(pre, dec, (2 * rank * g, (2 * rank + 1) * g), ((2 * rank + 1) * g, (2 * rank + 2) * g),
                       B.CORUN, sp, sd)
        torch.cuda.synchronize()
        bl.sync()
        out = (hp.cpu().numpy().copy(), hd.cpu().numpy().copy())
        dist.barrier()          # no rank unmaps a region a peer may still read
        if rank == 0:
            from harness import oracle_layer
            ref = oracle_layer(S, 0, S.x_pre.numpy(), S.x_dec.numpy())
            q.put((rank, out, (ref["pre"], ref["dec"])))
        else:
            q.put((rank, out, None))
        bl.close()
    finally:
        dist.destroy_process_group()


def test_peer_allreduce_two_processes_ipc():
    tp = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_rank, args=(r, tp, port, q)) for r in range(tp)]
    for p in ps:
        p.start()
    res = {}
    for _ in range(tp):
        r, out, ref = q.get(timeout=600)
        res[r] = (out, ref)
    for p in ps:
        p.join(120)
        assert p.exitcode == 0
    (o0, ref), (o1, _) = res[0], res[1]
    assert np.array_equal(o0[0], o1[0]) and np.array_equal(o0[1], o1[1])
    for got, want in zip(o0, ref):
        err = np.abs(got.astype(np.float64) - want)
        assert err.max() <= 2e-2 and err.sum() / np.abs(want).sum() <= 1e-3
