"""Fused tensor-parallel all-reduce over peer memory (PEER mode, SURVEY §8f
NEXT-2) on ONE B200: tp ranks are simulated by tp handles in this process,
each with its own Megatron weight / KV shard and its own SM ranges of the
same GPU (smid gating keeps the ranks' kernels on disjoint SMs, so their
fused GEMM + all-reduce kernels run at the same time and wait on each other
exactly as ranks on different GPUs would; the "peer" regions are local
memory instead of NVLink).  Checked against the unsharded CPU oracle layer,
per layer step (R-4c), with every rank's hidden bit-identical."""
import numpy as np
import pytest
import torch

from harness import Setup, compare, oracle_layer
from workload import synth

pytestmark = pytest.mark.gpu

M = synth.ModelShape("tp-sim", 1024, 8, 4, 128, 2048, 2)
PRE_LENS, DEC_CTX = [300, 77, 1], [64, 1, 500, 31, 16, 1000]


@pytest.fixture(scope="module")
def base():
    return Setup(M, PRE_LENS, DEC_CTX, n_layers=2)


def _ranks(S, tp):
    """tp PEER-mode handles (rank shards), connected to each other."""
    B = S.B
    from paper_conf_asplos_0001xc0l026_b200 import parallel
    lm = parallel.shard_model(B.Model.of(M), tp)
    ranks = []
    for r in range(tp):
        pools = [(parallel.shard_kv_pool(k, tp, r), parallel.shard_kv_pool(v, tp, r)) for k, v in S.pool_gpu]
        bl = B.Bullet(lm, pools, max_prefill_tokens=sum(PRE_LENS), max_decode_tokens=len(DEC_CTX),
                      max_position=S.bl_max_position if hasattr(S, "bl_max_position") else 2048,
                      tp_size=tp, tp_rank=r)
        for l in range(S.n_layers):
            bl.set_layer_weights(l, parallel.shard_layer_weights(S.w_gpu[l], B.Model.of(M), tp, r))
        ranks.append(bl)
    bases = [bl.tp_base() for bl in ranks]
    for bl in ranks:
        bl.tp_connect(bases)
    return ranks


def _batches(S, bl, x_pre, x_dec, lb, le):
    B = S.B
    bt = S.lay.block_table
    hp = bl.tp_hidden(0, x_pre.shape[0]); hp.copy_(x_pre)
    hd = bl.tp_hidden(1, x_dec.shape[0]); hd.copy_(x_dec)
    pre = B.Batch(PRE_LENS, [0] * len(PRE_LENS), bt[:S.n_pre], hp, lb, le)
    dec = B.Batch([1] * len(DEC_CTX), DEC_CTX, bt[S.n_pre:], hd, lb, le)
    return pre, dec


def _step_all(S, ranks, x_pre, x_dec, lb, le):
    """Every rank steps layers [lb, le) on its own SM ranges; returns each
    rank's (prefill, decode) hidden after the step."""
    tp = len(ranks)
    N = ranks[0].n_sms
    g = (N // (2 * tp)) & ~1
    cur = torch.cuda.current_stream()
    bs = [_batches(S, bl, x_pre, x_dec, lb, le) for bl in ranks]
    streams = []
    for r, bl in enumerate(ranks):
        sp, sd = torch.cuda.Stream(), torch.cuda.Stream()
        sp.wait_stream(cur); sd.wait_stream(cur)
        streams.append((sp, sd))
    for r, bl in enumerate(ranks):
        pre, dec = bs[r]
        bl.step_ranges(pre, dec, (2 * r * g, (2 * r + 1) * g), ((2 * r + 1) * g, (2 * r + 2) * g),
                       S.B.CORUN, *streams[r])
    torch.cuda.synchronize()
    for bl in ranks:
        bl.sync()   # surfaces a peer timeout
    return [(pre.hidden.clone(), dec.hidden.clone()) for pre, dec in bs]


@pytest.mark.parametrize("tp", [2, 4])
def test_peer_allreduce_layer_steps_match_oracle(base, tp):
    S = base
    ranks = _ranks(S, tp)
    x_pre, x_dec = S.x_pre.cuda(), S.x_dec.cuda()
    outs = []
    for l in range(2):
        got = _step_all(S, ranks, x_pre, x_dec, l, l + 1)
        for r in range(1, tp):   # every rank holds the same reduced residual stream
            assert torch.equal(got[r][0], got[0][0]) and torch.equal(got[r][1], got[0][1]), (tp, l, r)
        ref = oracle_layer(S, l, x_pre.cpu().numpy(), x_dec.cpu().numpy())
        for name, t in (("pre", got[0][0]), ("dec", got[0][1])):
            mx, mr = compare(t.cpu().numpy(), ref[name])
            assert mx <= 2e-2 and mr <= 1e-3, (tp, l, name, mx, mr)
        x_pre, x_dec = got[0]
        outs.append(got[0])
    # one 2-layer step == the two 1-layer steps, bit for bit (fixed reduction
    # order; the counters' expected values carried across steps)
    got2 = _step_all(S, ranks, S.x_pre.cuda(), S.x_dec.cuda(), 0, 2)
    assert torch.equal(got2[0][0], outs[1][0]) and torch.equal(got2[0][1], outs[1][1])
    for bl in ranks:
        bl.close()


def test_peer_mode_errors(base):
    S = base
    B = S.B
    from paper_conf_asplos_0001xc0l026_b200 import parallel
    lm = parallel.shard_model(B.Model.of(M), 2)
    pools = [(parallel.shard_kv_pool(k, 2, 0), parallel.shard_kv_pool(v, 2, 0)) for k, v in S.pool_gpu]
    bl = B.Bullet(lm, pools, max_prefill_tokens=sum(PRE_LENS), max_decode_tokens=len(DEC_CTX),
                  max_position=2048, tp_size=2, tp_rank=0)
    for l in range(2):
        bl.set_layer_weights(l, parallel.shard_layer_weights(S.w_gpu[l], B.Model.of(M), 2, 0))
    pre, dec = _batches(S, bl, S.x_pre.cuda(), S.x_dec.cuda(), 0, 1)
    with pytest.raises(B.BulletError) as e:      # not connected yet
        bl.step_ranges(pre, dec, (0, 74), (74, 148))
    assert e.value.code == -1
    with pytest.raises(B.BulletError):           # own base must sit at tp_rank
        bl.tp_connect([0x1000, bl.tp_base()])
    bl.tp_connect([bl.tp_base(), bl.tp_base()])
    wrong = B.Batch(PRE_LENS, [0] * len(PRE_LENS), S.lay.block_table[:S.n_pre], S.x_pre.cuda().contiguous(), 0, 1)
    with pytest.raises(B.BulletError) as e:      # hidden must be the symmetric buffer
        bl.step_ranges(wrong, None, (0, 74), (74, 148))
    assert e.value.code == -1
    assert len(bl.tp_ipc_handle()) == 64
    bl.close()
