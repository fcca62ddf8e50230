"""bullet_step parity (co-run prefill + decode layer step) vs the CPU oracle,
SM-gating invariants from the smid log, and error paths.  Needs a B200."""
import numpy as np
import pytest
import torch

from workload import synth
from harness import Setup, compare, phase_streams
from oracle import perfmodel as PM

pytestmark = pytest.mark.gpu


def _run(S, p, flags):
    B = S.B
    pre, dec = S.batches()
    sp, sd = phase_streams()
    S.bl.step(pre, dec, p, flags, sp, sd)
    torch.cuda.synchronize()
    return pre, dec


@pytest.fixture(scope="module")
def tiny():
    """BASELINE config 1: tiny 2-layer fp32 model, 1 x 128 prefill + 4 decodes
    with 64 cached tokens, paged KV block 16 (DESIGN R-6, R-7)."""
    wl = synth.workload("tiny")
    S = Setup(synth.MODELS["tiny"], wl.prefill_lens, wl.decode_ctx, n_layers=2)
    return S, S.oracle()


@pytest.mark.parametrize("mode", ["corun", "timesliced", "ungated"])
def test_tiny_fp32_two_layers(tiny, mode):
    S, ref = tiny
    B = S.B
    flags = {"corun": B.CORUN, "timesliced": B.TIMESLICED, "ungated": B.UNGATED}[mode]
    pre, dec = _run(S, 74, flags)
    for name, b in (("pre", pre), ("dec", dec)):
        mx, mr = compare(b.hidden.cpu().numpy(), ref[name])
        assert mx <= 1e-4 and mr <= 1e-5, (name, mx, mr)


@pytest.fixture(scope="module")
def small_bf16():
    m = synth.ModelShape("small-bf16", 1024, 8, 2, 128, 2816, 2)
    return Setup(m, [300, 77, 1], [64, 1, 500, 31, 16, 1000], n_layers=2)


def _per_layer(S, p, flags):
    """Run the two layers as two steps; check each step against the oracle
    layer fed with the GPU's own input to that step (R-4c), then check the
    single 2-layer step is bit-identical to the two 1-layer steps."""
    from harness import oracle_layer
    pre, dec = S.batches(0, 1)
    x_pre0, x_dec0 = pre.hidden.cpu().numpy(), dec.hidden.cpu().numpy()
    sp, sd = phase_streams()
    outs = []
    for l in range(2):
        pre.layer_begin, pre.layer_end = l, l + 1
        dec.layer_begin, dec.layer_end = l, l + 1
        xi_pre, xi_dec = pre.hidden.cpu().numpy(), dec.hidden.cpu().numpy()
        S.bl.step(pre, dec, p, flags, sp, sd)
        torch.cuda.synchronize()
        ref = oracle_layer(S, l, xi_pre, xi_dec)
        for name, b in (("pre", pre), ("dec", dec)):
            mx, mr = compare(b.hidden.cpu().numpy(), ref[name])
            assert mx <= 2e-2 and mr <= 1e-3, (name, l, p, mx, mr)
        outs.append((pre.hidden.clone(), dec.hidden.clone()))
    pre2, dec2 = S.batches(0, 2)
    S.bl.step(pre2, dec2, p, flags, sp, sd)
    torch.cuda.synchronize()
    assert torch.equal(pre2.hidden, outs[1][0]) and torch.equal(dec2.hidden, outs[1][1])


@pytest.mark.parametrize("p", [2, 64, 146])
def test_small_bf16_corun_splits(small_bf16, p):
    """Reduced Llama-style bf16 model (hd 128, GQA 4), two layer steps,
    ragged prefill lengths: co-run at edge and middle splits meets the bar."""
    _per_layer(small_bf16, p, small_bf16.B.CORUN)


@pytest.mark.parametrize("mode", ["timesliced", "ungated"])
def test_small_bf16_baseline_modes(small_bf16, mode):
    B = small_bf16.B
    _per_layer(small_bf16, 148, B.TIMESLICED if mode == "timesliced" else B.UNGATED)


def test_llama8b_config2_layer_sampled():
    """BASELINE config 2 at full Llama-3.1-8B layer dims (8 ShareGPT-shaped
    prefills summing to 4096 tokens + 128 decodes with 512-1536 cached
    tokens), one layer, the launch configuration bench.py times (co-run at
    the default split).  Oracle: all 128 decode rows and 64 sampled prefill
    rows incl. the last row of every request."""
    wl = synth.workload("sharegpt-8b")
    S = Setup(synth.MODELS["llama3.1-8b"], wl.prefill_lens, wl.decode_ctx, n_layers=1)
    n_p = sum(wl.prefill_lens)
    rng = np.random.default_rng(0)
    mask = np.zeros(n_p, np.uint8)
    mask[rng.choice(n_p, 48, replace=False)] = 1
    mask[np.cumsum(wl.prefill_lens) - 1] = 1
    ref = S.oracle(row_mask_pre=mask)
    pre, dec = _run(S, 104, S.B.CORUN)
    mx, mr = compare(dec.hidden.cpu().numpy(), ref["dec"])
    assert mx <= 2e-2 and mr <= 1e-3, ("dec", mx, mr)
    got = pre.hidden.cpu().numpy()[mask == 1]
    mx, mr = compare(got, ref["pre"][mask == 1])
    assert mx <= 2e-2 and mr <= 1e-3, ("pre", mx, mr)


def test_llama8b_config3_layer_sampled():
    """BASELINE config 3 at full size (one 8192-token arXiv-shaped prefill +
    256 decodes with 2048-6144 cached tokens, 5.4 GB of paged KV per layer),
    one layer at the split bench.py uses for it (p = 88).  Oracle: all 256
    decode rows and 49 sampled prefill rows incl. the last."""
    wl = synth.workload("arxiv-8b")
    S = Setup(synth.MODELS["llama3.1-8b"], wl.prefill_lens, wl.decode_ctx, n_layers=1)
    n_p = sum(wl.prefill_lens)
    rng = np.random.default_rng(1)
    mask = np.zeros(n_p, np.uint8)
    mask[rng.choice(n_p, 48, replace=False)] = 1
    mask[np.cumsum(wl.prefill_lens) - 1] = 1
    ref = S.oracle(row_mask_pre=mask)
    pre, dec = _run(S, 88, S.B.CORUN)
    mx, mr = compare(dec.hidden.cpu().numpy(), ref["dec"])
    assert mx <= 2e-2 and mr <= 1e-3, ("dec", mx, mr)
    got = pre.hidden.cpu().numpy()[mask == 1]
    mx, mr = compare(got, ref["pre"][mask == 1])
    assert mx <= 2e-2 and mr <= 1e-3, ("pre", mx, mr)


@pytest.mark.parametrize("p", [64, 146])
def test_fused_norm_bit_identical_to_rmsnorm_kernel(small_bf16, p):
    """RMSNorm in the O-proj / down GEMM tails (S6 and the next layer's S1)
    reproduces the standalone k_rmsnorm bit for bit (same reduction order)
    over a 2-layer step with ragged prefill rows, and launches 2 kernels
    fewer per layer after the first."""
    S = small_bf16
    B = S.B
    outs, launches = [], []
    for flags in (B.CORUN, B.CORUN | B.UNFUSED_NORM):
        pre, dec = S.batches(0, 2)
        sp, sd = phase_streams()
        n0 = S.bl.launch_count()
        S.bl.step(pre, dec, p, flags, sp, sd)
        torch.cuda.synchronize()
        launches.append(S.bl.launch_count() - n0)
        outs.append((pre.hidden.clone(), dec.hidden.clone()))
    assert torch.equal(outs[0][0], outs[1][0]) and torch.equal(outs[0][1], outs[1][1])
    # both batches have <= 1024 rows: 2 phases x (S6 x 2 layers + S1 of layer 1)
    assert launches[1] - launches[0] == 2 * (2 * 2 - 1)


@pytest.mark.parametrize("p", [2, 40, 146])
def test_smid_gating_invariants(small_bf16, p):
    """SM-range work assignment (§8a SG), bit-exact invariants: every work
    unit of every launch ran exactly once, on an SM of its phase's range;
    ranges = sigma[0:p) / sigma[p:N) (oracle range function)."""
    S = small_bf16
    B = S.B
    log = S.bl.set_smid_log(400000)
    try:
        _run(S, p, B.CORUN | B.SMID_LOG)
        n = int(log[0].item())
        assert 0 < n <= 400000
        e = log[1:1 + 4 * n].view(n, 4).cpu().numpy()
    finally:
        S.bl.set_smid_log(None)
    sigma = S.bl.sm_order()
    pre_set, dec_set = map(set, PM.sm_ranges(p, sigma))
    for launch in np.unique(e[:, 0]):
        rows = e[e[:, 0] == launch]
        phase = rows[0, 3]
        assert np.all(rows[:, 3] == phase)
        units = rows[:, 1]
        assert len(np.unique(units)) == len(units), "unit executed twice"
        assert units.min() == 0 and units.max() == len(units) - 1, "unit skipped"
        allowed = pre_set if phase == 0 else dec_set
        assert set(rows[:, 2].tolist()) <= allowed, (launch, phase)


def test_decode_pause_and_errors(small_bf16):
    S = small_bf16
    B = S.B
    pre, dec = S.batches()
    x0 = dec.hidden.clone()
    S.bl.step(pre, dec, S.bl.n_sms, B.CORUN)          # p = N: decode paused
    torch.cuda.synchronize()
    assert torch.equal(dec.hidden, x0)
    with pytest.raises(B.BulletError) as e:
        S.bl.step(pre, dec, 0, B.CORUN)
    assert e.value.code == -4
    with pytest.raises(B.BulletError) as e:
        S.bl.step(pre, dec, 3, B.CORUN)
    assert e.value.code == -4
    bad = S.lay.block_table[S.n_pre:].copy()
    bad[0, 0] = S.lay.n_blocks + 5
    dec_bad = B.Batch([1] * len(S.decode_ctx), S.decode_ctx, bad, dec.hidden)
    with pytest.raises(B.BulletError) as e:
        S.bl.step(None, dec_bad, 0, B.CORUN)
    assert e.value.code == -5
    # BULLET_CHECK_KV: disjoint prefill / decode block sets pass,
    # a decode request pointing at a prefill request's block is rejected
    S.bl.step(pre, dec, 64, B.CORUN | B.CHECK_KV)
    torch.cuda.synchronize()
    shared = S.lay.block_table[S.n_pre:].copy()
    shared[0, 0] = S.lay.block_table[0, 0]
    dec_sh = B.Batch([1] * len(S.decode_ctx), S.decode_ctx, shared, dec.hidden)
    with pytest.raises(B.BulletError) as e:
        S.bl.step(pre, dec_sh, 64, B.CORUN | B.CHECK_KV)
    assert e.value.code == -5


@pytest.mark.parametrize("bias", [0, 1])
@pytest.mark.parametrize("p", [40, 0])
def test_fused_qkv_rope_matches_unfused(p, bias):
    """S3 (RoPE + paged KV append) in the QKV GEMM epilogue (EPI_QKV) against
    the separate k_rope_kv kernel (BULLET_UNFUSED): same q, same pool
    contents (the only difference allowed is FMA contraction: <= 1 bf16 ulp),
    and both layer outputs meet the oracle bar."""
    m = synth.ModelShape("small-bias", 1024, 8, 2, 128, 2816, 1, qkv_bias=bias, rope_theta=1e6,
                         rope_llama3=0)
    S = Setup(m, [300, 77, 1, 129], [64, 1, 500, 31, 16], n_layers=1)
    ref = S.oracle()
    res = []
    mode = S.B.CORUN if p else S.B.TIMESLICED   # p = 0: both phases on all SMs
    p = p or S.bl.n_sms
    for flags in (mode | S.B.UNFUSED, mode):
        for k, v in S.pool_gpu:   # same starting pools
            k.zero_(); v.zero_()
        for (k, v), (kc, vc) in zip(S.pool_gpu, S.pool_cpu):
            k.copy_(kc.to(k.dtype)); v.copy_(vc.to(v.dtype))
        pre, dec = _run(S, p, flags)
        for name, b in (("pre", pre), ("dec", dec)):
            mx, mr = compare(b.hidden.cpu().numpy(), ref[name])
            assert mx <= 2e-2 and mr <= 1e-3, (flags, name, mx, mr)
        res.append((pre.hidden.clone(), dec.hidden.clone(), S.pool_gpu[0][0].clone(), S.pool_gpu[0][1].clone()))
    (a_pre, a_dec, a_k, a_v), (b_pre, b_dec, b_k, b_v) = res
    assert torch.equal(a_v, b_v)   # v: bias + bf16 round only, no rotation
    dk = (a_k.float() - b_k.float()).abs()
    assert float((dk / b_k.float().abs().clamp_min(1e-30)).max()) <= 2 ** -7
    assert float((a_pre - b_pre).abs().max()) <= 2e-2 and float((a_dec - b_dec).abs().max()) <= 2e-2


@pytest.mark.parametrize("bias", [0, 1])
def test_fused_qkv_pool_vs_oracle(bias):
    """S3 in the QKV GEMM epilogue (EPI_QKV, the default bf16 path) against
    the oracle directly: after one co-run layer step the pool holds the
    oracle's k / v at exactly the slots the definition names
    (block_table[r][p / 16] * 16 + p % 16 for every new position p of every
    request; a sentinel planted there must be gone), every other slot of the
    pool is bit-for-bit what it was, and the written values equal the
    oracle's R2-rounded k / v except for rare one-step rounding flips."""
    m = synth.ModelShape("qkvpool", 1024, 8, 2, 128, 2816, 1, qkv_bias=bias, rope_theta=1e6, rope_llama3=0)
    pre_lens, dec_ctx = [300, 77, 1, 129], [64, 1, 500, 31, 16, 0]
    S = Setup(m, pre_lens, dec_ctx, n_layers=1)
    q = pre_lens + [1] * len(dec_ctx)
    c = [0] * len(pre_lens) + dec_ctx
    slots = set()
    for r, (ql, cl) in enumerate(zip(q, c)):
        for i in range(ql):
            pos = cl + i
            slots.add((int(S.lay.block_table[r][pos // 16]), pos % 16))
    SENT = float("nan")   # a value no k / v can take
    for k, v in S.pool_cpu:                       # sentinel at every slot the step must write
        for blk, off in slots:
            k[blk, :, off, :] = SENT; v[blk, :, off, :] = SENT
    for (k, v), (kc, vc) in zip(S.pool_gpu, S.pool_cpu):
        k.copy_(kc.to(k.dtype)); v.copy_(vc.to(v.dtype))
    before_k, before_v = S.pool_cpu[0][0].clone(), S.pool_cpu[0][1].clone()
    # oracle: one layer on copies of the same pool (it writes k / v in place)
    import oracle as O
    from harness import oracle_cfg
    cfg = oracle_cfg(m)
    w = {kk: (None if vv is None else vv.numpy()) for kk, vv in S.w_cpu[0].items()}
    pk, pv = before_k.numpy().astype(np.float32).copy(), before_v.numpy().astype(np.float32).copy()
    O.layer_forward(cfg, w, pk, pv, pre_lens, [0] * len(pre_lens), S.lay.block_table[:S.n_pre],
                    S.x_pre.double().numpy())
    O.layer_forward(cfg, w, pk, pv, [1] * len(dec_ctx), dec_ctx, S.lay.block_table[S.n_pre:],
                    S.x_dec.double().numpy())
    _run(S, 64, S.B.CORUN)
    gk, gv = S.pool_gpu[0][0].float().cpu().numpy(), S.pool_gpu[0][1].float().cpu().numpy()
    mask = np.zeros((S.lay.n_blocks, 16), bool)
    for blk, off in slots:
        mask[blk, off] = True
    for got, ref, old in ((gk, pk, before_k.numpy()), (gv, pv, before_v.numpy())):
        g_s, r_s, o_s = (a.transpose(0, 2, 1, 3) for a in (got, ref, old))   # [blk][slot][Hkv][hd]
        assert np.array_equal(g_s[~mask], o_s[~mask])          # untouched slots: bit-identical
        assert not np.any(np.isnan(g_s[mask]))                # every named slot written
        gw, rw = g_s[mask].astype(np.float64), r_s[mask].astype(np.float64)   # oracle: already R2-rounded
        # equal, or one bf16 step apart (an R2 rounding flip); plus, for values
        # near 0, what an R1 flip of the token's normed input moves them by
        # (one bf16 step of h_i times |w_ij|: up to ~5e-4 per flipped h_i at d = 1024)
        bad = np.abs(gw - rw) > np.abs(rw) * 2.0 ** -7 + 2e-3
        assert not bad.any(), (int(bad.sum()), gw[bad][:8], rw[bad][:8], np.argwhere(bad)[:4])
        assert np.mean(gw == rw) > 0.99


@pytest.mark.parametrize("mode", ["timesliced", "corun"])
def test_hybrid_chunked_prefill_batch(mode):
    """Chunked-prefill hybrid batch: prefill chunks
    with cached context (ctx > 0, attention over the earlier chunks through the
    block table) followed by decode requests, as ONE batch through one layer:
    tcgen05 prefill attention over the chunks, decode kernel over the rest.
    Checked against the oracle layer on the same mixed batch."""
    from harness import oracle_cfg
    import oracle as O
    m = synth.ModelShape("small-bf16", 1024, 8, 2, 128, 2816, 1)
    q = [256, 130, 64, 1, 1, 1, 1, 1]
    c = [512, 77, 0, 63, 500, 16, 1000, 1]
    lay = synth.paged_layout(q, c, 16)
    w_cpu = synth.layer_weights(m, 0)
    pk_cpu, pv_cpu = synth.kv_pool(m, lay.n_blocks, 16, 0)
    x = synth.hidden(sum(q), m.d_model, seed_offset=0)
    import paper_conf_asplos_0001xc0l026_b200 as B
    pools = [(pk_cpu.to("cuda", torch.bfloat16).contiguous(), pv_cpu.to("cuda", torch.bfloat16).contiguous())]
    bl = B.Bullet(B.Model.of(m), pools, sum(q), 16, max(a + b for a, b in zip(q, c)) + 16)
    bl.set_layer_weights(0, {k: (None if v is None else v.to("cuda", torch.bfloat16)) for k, v in w_cpu.items()})
    b = B.Batch(q, c, lay.block_table, x.cuda().contiguous(), 0, 1)
    sp, sd = phase_streams()
    flags = B.TIMESLICED if mode == "timesliced" else B.CORUN
    bl.step(b, None, bl.n_sms if mode == "timesliced" else 64, flags, sp, sd)
    torch.cuda.synchronize()
    w = {k: (None if v is None else v.numpy()) for k, v in w_cpu.items()}
    ref = O.layer_forward(oracle_cfg(m), w, pk_cpu.numpy().copy(), pv_cpu.numpy().copy(), q, c,
                          lay.block_table, x.double().numpy())
    mx, mr = compare(b.hidden.cpu().numpy(), ref)
    assert mx <= 2e-2 and mr <= 1e-3, (mx, mr)
    n_pre = sum(q[:3])
    mx, mr = compare(b.hidden.cpu().numpy()[n_pre:], ref[n_pre:])   # the decode rows alone
    assert mx <= 2e-2 and mr <= 1e-3, ("decode rows", mx, mr)


@pytest.mark.parametrize("ranges", [((0, 80), (60, 148)), ((0, 148), (0, 148)), ((20, 100), (0, 40))])
def test_step_ranges_overlapping(small_bf16, ranges):
    """bullet_step_ranges (NEXT-4: non-strict partitions): with overlapping
    SM ranges both phases still meet the oracle bar, every unit runs exactly
    once, and each phase's units ran only inside its own range."""
    S = small_bf16
    B = S.B
    (plo, phi), (dlo, dhi) = ranges
    ref = S.oracle(layers=1)
    pre, dec = S.batches(0, 1)
    log = S.bl.set_smid_log(400000)
    try:
        sp, sd = phase_streams()
        S.bl.step_ranges(pre, dec, (plo, phi), (dlo, dhi), B.CORUN | B.SMID_LOG, sp, sd)
        torch.cuda.synchronize()
        n = int(log[0].item())
        e = log[1:1 + 4 * n].view(n, 4).cpu().numpy()
    finally:
        S.bl.set_smid_log(None)
    for name, b in (("pre", pre), ("dec", dec)):
        mx, mr = compare(b.hidden.cpu().numpy(), ref[name])
        assert mx <= 2e-2 and mr <= 1e-3, (name, mx, mr)
    sigma = list(S.bl.sm_order())
    allowed = {0: set(sigma[plo:phi]), 1: set(sigma[dlo:dhi])}
    for launch in np.unique(e[:, 0]):
        rows = e[e[:, 0] == launch]
        units = rows[:, 1]
        assert len(np.unique(units)) == len(units) and units.max() == len(units) - 1
        assert set(rows[:, 2].tolist()) <= allowed[int(rows[0, 3])]
    with pytest.raises(B.BulletError):
        S.bl.step_ranges(pre, dec, (0, 0), (0, 148), B.CORUN)   # non-empty batch, empty range


def test_cuda_graph_replay_matches_stream_launch(small_bf16):
    """NEXT-4: a co-run step captured into a CUDA graph (both phase streams
    forked from the capture stream) replays to the same bits as the direct
    launch: the per-step plan kernel re-zeroes the work counters and the split-K
    semaphores reset themselves, so replays are self-contained."""
    S = small_bf16
    B = S.B
    pre, dec = S.batches(0, 2)
    x_pre, x_dec = pre.hidden.clone(), dec.hidden.clone()
    sp, sd = phase_streams()

    def enqueue():
        ev = torch.cuda.Event(); ev.record(sp); sd.wait_event(ev)
        S.bl.step(pre, dec, 64, B.CORUN, sp, sd)
        ev2 = torch.cuda.Event(); ev2.record(sd); sp.wait_event(ev2)

    enqueue()
    torch.cuda.synchronize()
    want = (pre.hidden.clone(), dec.hidden.clone())
    g = torch.cuda.CUDAGraph()
    pre.hidden.copy_(x_pre); dec.hidden.copy_(x_dec)
    torch.cuda.synchronize()
    with torch.cuda.graph(g, stream=sp):
        enqueue()
    for _ in range(2):   # capture does not execute; every replay restarts from the inputs
        pre.hidden.copy_(x_pre); dec.hidden.copy_(x_dec)
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()
        assert torch.equal(pre.hidden, want[0]) and torch.equal(dec.hidden, want[1])


def test_device_split_graph_follows_set_split(small_bf16):
    """NEXT-4 with the split in device memory: one graph captured from a
    BULLET_DEVICE_SPLIT step at p = 64 replays at p = 100 after
    bullet_set_split — every unit runs inside the NEW ranges (smid log), and
    the bits equal the p = 64 replay (the captured GEMM plans fix the
    arithmetic; the split only moves where units run)."""
    S = small_bf16
    B = S.B
    pre, dec = S.batches(0, 2)
    x_pre, x_dec = pre.hidden.clone(), dec.hidden.clone()
    sp, sd = phase_streams()
    log = S.bl.set_smid_log(400000)
    sigma = list(S.bl.sm_order())

    def enqueue():
        ev = torch.cuda.Event(); ev.record(sp); sd.wait_event(ev)
        S.bl.step(pre, dec, 64, B.CORUN | B.DEVICE_SPLIT | B.SMID_LOG, sp, sd)
        ev2 = torch.cuda.Event(); ev2.record(sd); sp.wait_event(ev2)

    try:
        # direct DEVICE_SPLIT step == plain step at the same split
        S.bl.set_split((0, 64), (64, 148), sp)
        enqueue()
        torch.cuda.synchronize()
        direct = (pre.hidden.clone(), dec.hidden.clone())
        pre.hidden.copy_(x_pre); dec.hidden.copy_(x_dec)
        torch.cuda.synchronize()
        S.bl.step(pre, dec, 64, B.CORUN, sp, sd)
        torch.cuda.synchronize()
        assert torch.equal(pre.hidden, direct[0]) and torch.equal(dec.hidden, direct[1])
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=sp):
            enqueue()
        outs = []
        for p in (64, 100):
            pre.hidden.copy_(x_pre); dec.hidden.copy_(x_dec)
            S.bl.set_split((0, p), (p, 148), sp)
            log.zero_()
            torch.cuda.synchronize()
            g.replay()
            torch.cuda.synchronize()
            outs.append((pre.hidden.clone(), dec.hidden.clone()))
            n = int(log[0].item())
            e = log[1:1 + 4 * n].view(n, 4).cpu().numpy()
            allowed = {0: set(sigma[0:p]), 1: set(sigma[p:148])}
            assert n > 0
            for ph in (0, 1):
                rows = e[e[:, 3] == ph]
                assert set(rows[:, 2].tolist()) <= allowed[ph], (p, ph)
        assert torch.equal(outs[0][0], outs[1][0]) and torch.equal(outs[0][1], outs[1][1])
        assert torch.equal(outs[0][0], direct[0]) and torch.equal(outs[0][1], direct[1])
    finally:
        S.bl.set_smid_log(None)


def test_pdl_on_off_bit_identical():
    """Programmatic dependent launch changes when kernels start, never what
    they compute: a two-layer co-run step with PDL (default) and without
    (BULLET_PDL=0, fresh process) gives the same bits."""
    import os
    import subprocess
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    code = ("import sys; sys.path[:0] = [%r, %r]\n"
            "import torch, hashlib\n"
            "from harness import Setup, phase_streams\n"
            "from workload import synth\n"
            "m = synth.ModelShape('pdl', 1024, 8, 2, 128, 2816, 2)\n"
            "S = Setup(m, [300, 77, 1], [64, 1, 500, 31], n_layers=2)\n"
            "pre, dec = S.batches()\n"
            "S.bl.step(pre, dec, 64, S.B.CORUN, *phase_streams())\n"
            "torch.cuda.synchronize()\n"
            "h = hashlib.sha256(pre.hidden.cpu().numpy().tobytes() + dec.hidden.cpu().numpy().tobytes())\n"
            "print('DIGEST', h.hexdigest())\n") % (here, os.path.dirname(here))
    digests = []
    for pdl in ("1", "0"):
        r = subprocess.run([sys.executable, "-c", code], env=dict(os.environ, BULLET_PDL=pdl),
                           capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-3000:]
        digests.append([l for l in r.stdout.splitlines() if l.startswith("DIGEST")][0])
    assert digests[0] == digests[1]


def test_prefill_attention_gqa_pair_bit_identical():
    """Two query heads of a GQA group per CTA (k_attn_prefill5<2>, the
    default for even group sizes) change which CTA computes a head, never the
    per-row arithmetic: a two-layer co-run step with ragged prompts (partial
    query tiles, a 1-token prompt) gives the same bits as the one-head kernel
    (BULLET_PF5_NQ=1, fresh process)."""
    import os
    import subprocess
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    code = ("import sys; sys.path[:0] = [%r, %r]\n"
            "import torch, hashlib\n"
            "from harness import Setup, phase_streams\n"
            "from workload import synth\n"
            "m = synth.ModelShape('gqa', 1024, 8, 2, 128, 2816, 2)\n"
            "S = Setup(m, [300, 77, 1, 129], [64, 1, 500, 31], n_layers=2)\n"
            "pre, dec = S.batches()\n"
            "S.bl.step(pre, dec, 64, S.B.CORUN, *phase_streams())\n"
            "torch.cuda.synchronize()\n"
            "h = hashlib.sha256(pre.hidden.cpu().numpy().tobytes() + dec.hidden.cpu().numpy().tobytes())\n"
            "print('DIGEST', h.hexdigest())\n") % (here, os.path.dirname(here))
    digests = []
    for nq in ("0", "1"):
        r = subprocess.run([sys.executable, "-c", code], env=dict(os.environ, BULLET_PF5_NQ=nq),
                           capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-3000:]
        digests.append([l for l in r.stdout.splitlines() if l.startswith("DIGEST")][0])
    assert digests[0] == digests[1]


def test_prefill_attention_tma_kv_bit_identical():
    """K / V tiles fed by TMA (the default: a full 64-key tile is 8 boxes of
    16 pool rows x 64 dims, 128-byte swizzle) land in the same swizzled
    shared-memory layout as the cp.async gathers: a two-layer co-run step with
    ragged prompts (full tiles, partial last tiles, a 1-token prompt, a
    16-aligned prompt) gives the same bits with BULLET_PF5_TMA=0 (every tile
    gathered by cp.async, fresh process), for both the GQA-pair and the
    one-head kernel."""
    import os
    import subprocess
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    code = ("import sys; sys.path[:0] = [%r, %r]\n"
            "import torch, hashlib\n"
            "from harness import Setup, phase_streams\n"
            "from workload import synth\n"
            "m = synth.ModelShape('gqa', 1024, 8, 2, 128, 2816, 2)\n"
            "S = Setup(m, [300, 77, 1, 129, 256], [64, 1, 500, 31], n_layers=2)\n"
            "pre, dec = S.batches()\n"
            "S.bl.step(pre, dec, 64, S.B.CORUN, *phase_streams())\n"
            "torch.cuda.synchronize()\n"
            "h = hashlib.sha256(pre.hidden.cpu().numpy().tobytes() + dec.hidden.cpu().numpy().tobytes())\n"
            "print('DIGEST', h.hexdigest())\n") % (here, os.path.dirname(here))
    for nq in ("0", "1"):
        digests = []
        for tma in ("1", "0"):
            r = subprocess.run([sys.executable, "-c", code],
                               env=dict(os.environ, BULLET_PF5_TMA=tma, BULLET_PF5_NQ=nq),
                               capture_output=True, text=True, timeout=600)
            assert r.returncode == 0, r.stderr[-3000:]
            digests.append([l for l in r.stdout.splitlines() if l.startswith("DIGEST")][0])
        assert digests[0] == digests[1], nq


@pytest.mark.parametrize("knob", ["BULLET_GEMM_EPI_COAL=0", "BULLET_DEC_TMA=0"])
def test_layout_knobs_bit_identical(knob):
    """Round-2 data-movement changes that must not touch the arithmetic: the
    GEMM epilogues' shared-memory transposed loads / stores (off:
    BULLET_GEMM_EPI_COAL=0, per-row vectors) and the decode attention's TMA
    stream (off: BULLET_DEC_TMA=0, cp.async) — a two-layer co-run step with
    ragged prompts and decodes gives the same bits either way (fresh
    processes)."""
    import os
    import subprocess
    import sys
    here = os.path.dirname(os.path.abspath(__file__))
    code = ("import sys; sys.path[:0] = [%r, %r]\n"
            "import torch, hashlib\n"
            "from harness import Setup, phase_streams\n"
            "from workload import synth\n"
            "m = synth.ModelShape('gqa', 1024, 8, 2, 128, 2816, 2)\n"
            "S = Setup(m, [300, 77, 1, 129, 256], [64, 1, 500, 31, 2047, 16], n_layers=2)\n"
            "pre, dec = S.batches()\n"
            "S.bl.step(pre, dec, 64, S.B.CORUN, *phase_streams())\n"
            "torch.cuda.synchronize()\n"
            "h = hashlib.sha256(pre.hidden.cpu().numpy().tobytes() + dec.hidden.cpu().numpy().tobytes())\n"
            "print('DIGEST', h.hexdigest())\n") % (here, os.path.dirname(here))
    k, v = knob.split("=")
    digests = []
    for env in ({}, {k: v}):
        r = subprocess.run([sys.executable, "-c", code], env=dict(os.environ, **env),
                           capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stderr[-3000:]
        digests.append([l for l in r.stdout.splitlines() if l.startswith("DIGEST")][0])
    assert digests[0] == digests[1], knob
