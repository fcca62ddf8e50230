"""NEXT-1 serving loop (serving.py) on the host: the loop's bookkeeping
driven by the host-only performance model (bullet_perf_create) as the step
time and by the product's Alg. 1 (bullet_choose_split) as the split decision.
Checks the invariants a GPU run relies on: every request generates exactly
its tokens, KV blocks are all returned, prefill batches advance layer by
layer to the end, decode membership changes only between iterations, and
each policy's pausing rule holds."""
import json
import os

import pytest

from paper_conf_asplos_0001xc0l026_b200 import serving as SV
from paper_conf_asplos_0001xc0l026_b200.bullet import Model, PerfModel
from workload import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
L, N = 32, 148


@pytest.fixture(scope="module")
def pm():
    pj = os.path.join(ROOT, "profiles", "perf_params_b200.json")
    return PerfModel(Model.of(synth.MODELS["llama3.1-8b"]), N, open(pj).read() if os.path.exists(pj) else None)


class Recorder:
    """Step stand-in: model-predicted device time + a record of every call."""

    def __init__(self, pm):
        self.pm, self.calls = pm, []

    def __call__(self, pw, dw, p, mode):
        self.calls.append((pw, dw, p, mode,
                           None if pw is None else (pw.batch_id, pw.layer_begin, pw.layer_end, tuple(r.rid for r in pw.reqs)),
                           None if dw is None else (dw.batch_id, dw.layer_begin, dw.layer_end, tuple(r.rid for r in dw.reqs))))
        both = pw is not None and dw is not None and mode == "corun"
        tp = td = 0.0
        if pw is not None:
            sm = p if mode == "corun" else N
            tp = self.pm.predict_us(pw.q_lens, pw.ctx_lens, sm, N - sm if both else 0) * (pw.layer_end - pw.layer_begin)
        if dw is not None:
            sm = N - p if mode == "corun" else N
            td = self.pm.predict_us(dw.q_lens, dw.ctx_lens, sm, p if both else 0) * (dw.layer_end - dw.layer_begin)
        return (max(tp, td) if mode == "corun" else tp + td) / 1e3


def _run(pm, policy, rate=40.0, dur=1.0):
    trace = SV.poisson_trace(rate, dur, seed=3)
    rec = Recorder(pm)
    alloc = SV.BlockAllocator(8000)
    loop = SV.ServingLoop(L, N, rec, pm.choose_split, policy, alloc, max_decodes=128, k_full=4)
    res = loop.run(trace)
    return trace, rec, alloc, loop, res


@pytest.mark.parametrize("policy", ["bullet", "bullet_tput", "bullet_gain", "static", "timesliced", "prefill_first", "chunked"])
def test_every_request_completes_and_blocks_return(pm, policy):
    trace, rec, alloc, loop, res = _run(pm, policy)
    assert res["finished"] == len(trace) > 10
    for r in trace:
        assert r.tokens == r.out_len and r.finish_ms >= r.first_token_ms >= r.arrival_ms
    assert len(alloc.free) == alloc.n_blocks and sorted(alloc.free) == list(range(alloc.n_blocks))
    json.dumps(res)   # serialisable metrics


@pytest.mark.parametrize("policy", ["bullet", "timesliced", "prefill_first", "chunked"])
def test_layer_progress_and_decode_membership(pm, policy):
    trace, rec, alloc, loop, res = _run(pm, policy)
    pre, dec = {}, {}
    for *_, pinfo, dinfo in rec.calls:
        for info, seen in ((pinfo, pre), (dinfo, dec)):
            if info is None:
                continue
            bid, lb, le, rids = info
            s = seen.setdefault(bid, {"next": 0, "rids": rids})
            assert lb == s["next"] and lb < le <= L, (bid, lb, le, s)
            assert rids == s["rids"]          # membership fixed within a batch / iteration
            s["next"] = le
    # every prefill batch ran all layers; decode iterations other than the
    # last ones ran all layers too
    assert all(s["next"] == L for s in pre.values())
    assert sum(s["next"] == L for s in dec.values()) >= len(dec) - 1


def test_policy_rules(pm):
    _, rec, *_ = _run(pm, "prefill_first")
    assert all(dw is None for pw, dw, *_ in rec.calls if pw is not None)       # decode paused
    _, rec, *_ = _run(pm, "timesliced")
    assert all(mode == "timesliced" and p == N for pw, dw, p, mode, *_ in rec.calls)
    _, rec, *_ = _run(pm, "bullet")
    both = [(p, dw) for pw, dw, p, mode, *_ in rec.calls if pw is not None and dw is not None]
    assert both and all(0 < p < N for p, _ in both)                           # a real split
    assert all(p % 2 == 0 for pw, dw, p, mode, *_ in rec.calls)              # TPC granularity


def test_chunked_policy_batches():
    """Chunked prefill: every cycle is one hybrid batch on all SMs (prefill
    chunks with q > 1 first, then q = 1 rows), within the token budget; a
    prompt's chunks cover it exactly once, in order (ctx = tokens before)."""
    trace = SV.poisson_trace(40.0, 1.0, seed=3)
    rec = Recorder(pm_fixture_cache())
    loop = SV.ServingLoop(L, N, rec, None, "chunked", SV.BlockAllocator(8000), max_decodes=128, k_full=4,
                          chunk_tokens=512)
    loop.run(trace)
    covered = {}
    for pw, dw, p, mode, pinfo, _ in rec.calls:
        assert dw is None and mode == "timesliced" and p == N
        assert sum(pw.q_lens) <= max(512, sum(1 for q in pw.q_lens if q == 1))
        ones = [q == 1 for q in pw.q_lens]
        assert ones == sorted(ones)                     # q > 1 rows first
        if pw.layer_begin == 0:
            for r, q, c in zip(pw.reqs, pw.q_lens, pw.ctx_lens):
                if c < r.prompt:                        # a prefill chunk of r
                    assert covered.get(r.rid, 0) == c
                    covered[r.rid] = c + q
    assert all(covered[r.rid] == r.prompt for r in trace)


_PM = []


def pm_fixture_cache():
    if not _PM:
        pj = os.path.join(ROOT, "profiles", "perf_params_b200.json")
        _PM.append(PerfModel(Model.of(synth.MODELS["llama3.1-8b"]), N, open(pj).read() if os.path.exists(pj) else None))
    return _PM[0]


def test_trace_is_seeded_and_shaped():
    a, b = SV.poisson_trace(50, 2.0, seed=1), SV.poisson_trace(50, 2.0, seed=1)
    assert [(r.arrival_ms, r.prompt, r.out_len) for r in a] == [(r.arrival_ms, r.prompt, r.out_len) for r in b]
    assert 60 < len(a) < 140                                                 # ~100 arrivals
    assert all(32 <= r.prompt <= 2048 and 8 <= r.out_len <= 512 for r in a)


def test_online_feedback_learns_observed_contention():
    """P:L195 online estimator feedback: when every co-run cycle takes 1.3x
    what the model predicts (a fixed, uncorrected contention), the loop's EMA
    converges to that ratio and the model's co-location factors are rescaled
    by 1/1.3 — later co-run predictions match the observations; non-co-run
    predictions are untouched.  The factors are restored afterwards."""
    pj = os.path.join(ROOT, "profiles", "perf_params_b200.json")
    truth = PerfModel(Model.of(synth.MODELS["llama3.1-8b"]), N, open(pj).read())   # uncorrected
    est = PerfModel(Model.of(synth.MODELS["llama3.1-8b"]), N, open(pj).read())     # corrected online
    base = est.colocation()

    class Slow(Recorder):
        def __call__(self, pw, dw, p, mode):
            ms = super().__call__(pw, dw, p, mode)
            return ms * 1.3 if (pw is not None and dw is not None and mode == "corun" and 0 < p < N) else ms

    trace = SV.poisson_trace(60.0, 1.0, seed=5)
    loop = SV.ServingLoop(L, N, Slow(truth), est.choose_split, "bullet", SV.BlockAllocator(8000),
                          max_decodes=128, k_full=4, feedback_model=est)
    res = loop.run(trace)
    assert res["finished"] == len(trace)
    n_co = sum(1 for c in loop.log if 0 < c[1] < N and c[2] > 0 and c[3] > 0)
    assert n_co > 20
    assert abs(loop.fb_ratio - 1.3) < 0.02, loop.fb_ratio
    pc, pb = est.colocation()
    assert abs(pc - base[0] / loop.fb_ratio) < 1e-12 and abs(pb - base[1] / loop.fb_ratio) < 1e-12
    q, c = [512, 300], [0, 0]
    assert est.predict_us(q, c, 100, 48) == pytest.approx(truth.predict_us(q, c, 100, 48) * loop.fb_ratio, rel=1e-9)
    assert est.predict_us(q, c, 148, 0) == truth.predict_us(q, c, 148, 0)   # alone: no co-location factor
    est.set_colocation(*base)
    with pytest.raises(Exception):
        est.set_colocation(0.0, 1.0)


@pytest.mark.parametrize("policy", ["bullet", "timesliced", "prefill_first"])
def test_unservable_request_ends_the_loop(pm, policy):
    """A request whose prompt exceeds max_prefill_tokens can never be admitted:
    once the rest of the trace is served the loop stops and reports it (it
    never builds a prefill batch out of nothing)."""
    trace = SV.poisson_trace(40.0, 0.3, seed=3)
    big = SV.Request(rid=10 ** 6, arrival_ms=trace[-1].arrival_ms + 1.0, prompt=9000, out_len=4)
    rec = Recorder(pm)
    loop = SV.ServingLoop(L, N, rec, pm.choose_split, policy, SV.BlockAllocator(8000), max_decodes=128,
                          k_full=4, max_prefill_tokens=8192)
    res = loop.run(trace + [big])
    assert res["finished"] == len(trace) and res["unservable"] == 1 and loop.unservable[0].rid == 10 ** 6
