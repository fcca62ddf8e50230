"""Pins of oracle/perfmodel.py (Eq. 1, Eq. 2, T_m, Alg. 1 reading) against the
paper's printed numbers (Table 1; O-proj bound), closed forms
and brute-force enumeration.  CPU only."""
import json
import math
import os

import pytest

from oracle import perfmodel as PM

GOLD = os.path.join(os.path.dirname(__file__), "golden", "table1_wave_idle.json")


def test_eq1_reproduces_table1_columns():
    """Eq. 1 with the grid of each kernel reproduces the 12 reproducible
    Table 1 entries to the printed 0.1 %."""
    t = json.load(open(GOLD))
    M = t["M"]
    for row in t["rows"]:
        sl = row["sl"]
        got = {"QKV": PM.wave_idle((sl // 128) * (6144 // 256), M),
               "Attn": PM.wave_idle((sl // 128) * 32, M),
               "OProj": PM.wave_idle((sl // 128) * (4096 // 256), M)}
        for k, v in got.items():
            assert abs(100 * v - row[k]) <= 0.05 + 1e-9, (sl, k, 100 * v, row[k])


def test_oproj_theoretical_bound_consistency():
    """O-proj theoretical utilisation bound 59 % / 79 % = 1 - s."""
    t = json.load(open(GOLD))["oproj_theoretical_bound_pct"]
    for sl in (1024, 2048):
        s = PM.wave_idle((sl // 128) * 16, 108)
        assert round(100 * (1 - s)) == t[str(sl)]


def test_eq1_closed_forms():
    assert PM.wave_idle(148 * 3, 148) == 0.0
    assert math.isclose(PM.wave_idle(37, 148), 1 - 37 / 148)
    assert PM.wave_idle(0, 148) == 0.0
    assert math.isclose(PM.wave_idle(149, 148), 1 - 149 / 296)


def test_eq2_reduces_to_plain_roofline():
    """m = M, d = p = 1, s = 0 -> max(c/C, b/B)."""
    for c, b in [(1e12, 1e6), (1e6, 1e12), (3e9, 2e9)]:
        t = PM.kernel_time(c, b, 1e15, 1e12, 148, 148, 1, 1, 1, 1, 0.0)
        assert t == max(c / 1e15, b / 1e12)


def test_eq2_with_wave_quantization_closed_form():
    """Compute-bound kernel of g tiles, d = p = 1: Eq. 1 + Eq. 2 give
    t(m) = c/C * M * ceil(g/m) / g, which is non-increasing in m."""
    c, C, M, g = 2e12, 1.6e15, 148, 300
    prev = math.inf
    for m in range(2, 149, 2):
        t = PM.kernel_time(c, 0, C, 1, M, m, 1, 1, 1, 1, PM.wave_idle(g, m))
        assert math.isclose(t, c / C * M * math.ceil(g / m) / g, rel_tol=1e-12)
        assert t <= prev * (1 + 1e-12)
        prev = t


def test_layer_kernel_inventory_flops():
    """Flop counts of the inventory: GEMMs 2 n K N; attention 4 hd H x causal
    pairs, pairs = s(s+1)/2 per prefill request, ctx+1 per decode request."""
    P = PM.default_params()
    shape = dict(d=4096, H=32, Hkv=8, hd=128, I=14336, elt=2, q_lens=[512, 100], ctx_lens=[0, 0])
    ks = {k[0]: k for k in PM.layer_kernels(shape, P, 148)}
    n = 612
    # bf16 / hd 128: RoPE (6 flops per rotated pair element) rides in the QKV epilogue, no rope_kv kernel
    assert ks["qkv"][1] == 2.0 * n * 4096 * 6144 + 6.0 * n * (32 + 8) * 128
    assert ks["qkv"][2] == 2 * (4096 * 6144 + n * 4096) + 2 * n * 6144   # weights + A + bf16 q/k/v out
    assert "rope_kv" not in ks
    f32 = {k[0]: k for k in PM.layer_kernels(dict(shape, elt=4), P, 148)}
    assert f32["qkv"][1] == 2.0 * n * 4096 * 6144 and f32["rope_kv"][1] == 6.0 * n * (32 + 8) * 128
    assert ks["o_proj"][1] == 2.0 * n * 4096 * 4096
    assert ks["gate_up"][1] == 2.0 * n * 4096 * 2 * 14336
    assert ks["down"][1] == 2.0 * n * 14336 * 4096
    assert ks["attn"][1] == 4.0 * 128 * 32 * (512 * 513 // 2 + 100 * 101 // 2)
    dec = dict(shape, q_lens=[1] * 4, ctx_lens=[10, 20, 30, 40])
    kd = {k[0]: k for k in PM.layer_kernels(dec, P, 148)}
    assert kd["attn"][1] == 4.0 * 128 * 32 * (11 + 21 + 31 + 41)
    assert kd["attn"][2] == 2 * 2 * 8 * 128 * (11 + 21 + 31 + 41) + 2 * 2 * 4 * 32 * 128
    assert kd["attn"][3] == 4 * 8


def test_layer_time_monotone_in_sms():
    P = PM.default_params()
    shape = dict(d=4096, H=32, Hkv=8, hd=128, I=14336, elt=2, q_lens=[4096], ctx_lens=[0])
    ts = [PM.layer_time(shape, P, m, 0) for m in range(8, 149, 2)]
    # not strictly monotone under split-K re-planning, but close: within 2 %
    for a, b in zip(ts, ts[1:]):
        assert b <= a * 1.02


def test_interp_piecewise_linear():
    tab = {"m": [10, 20, 40], "v": [0.5, 0.7, 1.0]}
    assert PM.interp(tab, 5) == 0.5 and PM.interp(tab, 40) == 1.0 and PM.interp(tab, 100) == 1.0
    assert math.isclose(PM.interp(tab, 15), 0.6) and math.isclose(PM.interp(tab, 30), 0.85)


def test_p90_nearest_rank():
    assert PM.p90([]) == 0.0
    assert PM.p90(list(range(1, 11))) == 9
    assert PM.p90([5]) == 5
    assert PM.p90(list(range(1, 21))) == 18


def test_sm_ranges_partition():
    sigma = list(range(0, 296, 2))
    for p in (0, 2, 146, 148):
        a, b = PM.sm_ranges(p, sigma)
        assert len(a) == p and set(a).isdisjoint(b) and sorted(a + b) == sorted(sigma)


# -------------------------------------------------------------- Alg. 1

MODEL = dict(d=4096, H=32, Hkv=8, hd=128, I=14336, elt=2)
SLO = {"ttft_norm_ms_per_tok": 1.5, "tpot_ms": 175.0, "w_max": 4, "v_min": 16, "percentile": 0.9}


def _state(**kw):
    s = dict(layers_done=4, total_layers=32, prefill_lens=[2048], prefill_waited_ms=[100.0],
             pending_lens=[], pending_waited_ms=[], decode_tokens=[50] * 64,
             decode_elapsed_ms=[50 * 20.0] * 64, decode_mean_ctx=1024, u_k=100, v_k=48)
    s.update(kw)
    return s


def _eval_all(P, st, slo):
    return {v: PM.evaluate_split(P, MODEL, st, slo, P["M"] - v, v) for v in PM.candidates(P, slo, 2)}


def test_case_both_ok_reduces_decode_to_minimal_feasible():
    """Alg. 1 l.12-13: both SLOs met -> ReduceDecodeSM: the smallest decode SM
    count that still meets both SLOs (prefill priority)."""
    P = PM.default_params()
    st = _state()
    ev = _eval_all(P, st, SLO)
    assert ev[48][0] <= 1 and ev[48][1] <= 1
    u, k = PM.choose_split(P, MODEL, st, SLO)
    v = P["M"] - u
    assert ev[v][0] <= 1 and ev[v][1] <= 1
    assert all(not (ev[w][0] <= 1 and ev[w][1] <= 1) for w in ev if w < v)
    assert k >= 1


def test_objective_throughput_picks_feasible_split_with_most_tokens_per_ms():
    """R-21 (objective 1): both SLOs met -> among the SLO-feasible
    splits the one with the highest predicted (prefill tokens + decode tokens
    x k) / cycle, checked by brute force over every candidate; objective 0
    keeps Alg. 1's ReduceDecodeSM."""
    P = PM.default_params()
    st = _state()
    slo1 = dict(SLO, objective=1)
    ev = _eval_all(P, st, slo1)
    dec = PM._phase_shape(MODEL, [1] * 64, [1024] * 64)

    def tput(v):
        t_p, t_d = ev[v][2], PM.layer_time(dec, P, v, P["M"] - v) * 1e3
        k = max(1, int(math.floor(t_p / t_d + 0.5)))
        return (2048 + 64 * k) / max(t_p, k * t_d), k
    feas = [v for v in ev if ev[v][0] <= 1 and ev[v][1] <= 1]
    u, k = PM.choose_split(P, MODEL, st, slo1)
    v = P["M"] - u
    assert v in feas and tput(v)[0] == max(tput(w)[0] for w in feas) and k == tput(v)[1]
    u0, _ = PM.choose_split(P, MODEL, st, SLO)          # objective 0 unchanged: fewest decode SMs
    assert P["M"] - u0 == min(feas) and tput(P["M"] - u0)[0] <= tput(v)[0]


def test_objective_throughput_takes_timesliced_cycle_when_corun_costs_more():
    """R-22: with both SLOs met and co-location made expensive (p_c = p_b =
    0.3: every co-run kernel 3.3x slower), the time-sliced cycle (prefill layer
    then k_ts = round(t_p / t_d) decode layer-steps, all SMs each) has more
    predicted tokens/ms than any co-run split, so objective 1 returns it as
    (N, k_ts); with the fitted-free default factors co-running wins."""
    P = dict(PM.default_params(), p_c=0.3, p_b=0.3)
    st = _state()
    slo1 = dict(SLO, objective=1)
    N = P["M"]
    pre = PM._phase_shape(MODEL, [2048], [0])
    dec = PM._phase_shape(MODEL, [1] * 64, [1024] * 64)
    tp, td = PM.layer_time(pre, P, N, 0) * 1e3, PM.layer_time(dec, P, N, 0) * 1e3
    k_ts = max(1, int(math.floor(tp / td + 0.5)))
    t_ts = (2048 + 64 * k_ts) / (tp + k_ts * td)
    ev = _eval_all(P, st, slo1)
    t_co = 0.0
    for v, (a, b, t_p) in ev.items():
        if a <= 1 and b <= 1:
            t_d = PM.layer_time(dec, P, v, N - v) * 1e3
            k = max(1, int(math.floor(t_p / t_d + 0.5)))
            t_co = max(t_co, (2048 + 64 * k) / max(t_p, k * t_d))
    assert t_ts > t_co
    assert PM.choose_split(P, MODEL, st, slo1) == (N, k_ts)
    u, k = PM.choose_split(PM.default_params(), MODEL, st, slo1)
    assert u < N   # default factors: a co-run split


def test_case_both_violated_sets_balanced():
    """Alg. 1 l.15-16 (R-14): both violated -> argmin of max ratio."""
    P = PM.default_params()
    st = _state(prefill_waited_ms=[4000.0], decode_elapsed_ms=[50 * 400.0] * 64)
    ev = _eval_all(P, st, SLO)
    assert ev[48][0] > 1 and ev[48][1] > 1
    u, _ = PM.choose_split(P, MODEL, st, SLO)
    best = min(max(e[0], e[1]) for e in ev.values())
    assert max(ev[P["M"] - u][0], ev[P["M"] - u][1]) == best


def test_case_tpot_violated_reduces_prefill():
    """Alg. 1 l.18-19: TTFT ok, TPOT violated, queue short -> smallest decode
    increase that meets TPOT."""
    P = PM.default_params()
    st = _state(v_k=16, u_k=132, decode_tokens=[0] * 64, decode_elapsed_ms=[0.0] * 64,
                prefill_waited_ms=[0.0])
    slo = dict(SLO, tpot_ms=20.0)
    ev = _eval_all(P, st, slo)
    assert ev[16][0] <= 1 and ev[16][1] > 1
    u, _ = PM.choose_split(P, MODEL, st, slo)
    v = P["M"] - u
    assert v > 16 and ev[v][1] <= 1
    assert all(ev[w][1] > 1 for w in ev if 16 <= w < v)


def test_case_ttft_violated_pauses_decode_when_tpot_allows():
    """§3.3.3: TTFT violated even at v_min while TPOT holds ->
    pause decode for the cycle (prefill gets all SMs, k = 0)."""
    P = PM.default_params()
    st = _state(prefill_waited_ms=[3053.0], decode_elapsed_ms=[50 * 1.0] * 64)
    ev = _eval_all(P, st, SLO)
    assert all(e[0] > 1 for e in ev.values())
    assert PM.choose_split(P, MODEL, st, SLO) == (P["M"], 0)


def test_degenerate_states():
    P = PM.default_params()
    assert PM.choose_split(P, MODEL, _state(decode_tokens=[], decode_elapsed_ms=[]), SLO) == (148, 0)
    assert PM.choose_split(P, MODEL, _state(prefill_lens=[], prefill_waited_ms=[]), SLO) == (0, 32)


def test_fitted_model_heldout_report_reproduces():
    """The reported fit quality (profiles/r01c_perfmodel_eval.json: held-out
    MRE and SLO-classification accuracy) is what the committed
    parameters give on the committed B200 measurements with the host-only
    model of the product (bullet_perf_create) — no GPU needed."""
    import json
    import os
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, os.path.join(root, "scripts"))
    import fit_perfmodel as F
    pp = os.path.join(root, "profiles", "perf_params_b200.json")
    got = F.evaluate(pp, pp.replace(".json", "_points.json"))
    want = json.load(open(os.path.join(root, "profiles", "r02_perfmodel_eval.json")))
    assert abs(got["mre_heldout"] - want["mre_heldout"]) < 1e-9
    assert abs(got["slo_accuracy_heldout"] - want["slo_accuracy_heldout"]) < 1e-9
    assert got["mre_heldout"] < 0.191 and got["slo_accuracy_heldout"] > 0.88   # paper's numbers, context


# ------------------------------------------- Alg. 1 l.3-10, hand-derived pins
# evaluate_split and the R-21 / R-22 candidates are pinned here against values
# worked out by hand from Alg. 1 with a stub layer time, so a
# slip in rem_time, the queueing term, the TPOT update or the cycle / k
# arithmetic fails independently of the kernel inventory.  Stub (ms): prefill
# layer of n new tokens on m SMs = n / 3 / m, decode layer = 10 / m, both x f
# when a co-runner holds SMs (f = 1.25), and M = 100 SMs.

def _stub_layer_time(f):
    def lt(shape, P, m, corun_m):
        if m <= 0:
            return math.inf
        g = f if corun_m > 0 else 1.0
        q = shape["q_lens"]
        ms = 10.0 / m * g if all(x == 1 for x in q) else sum(q) / 3.0 / m * g
        return ms / 1e3
    return lt


HAND = dict(layers_done=4, total_layers=32, prefill_lens=[100, 200], prefill_waited_ms=[10.0, 20.0],
            pending_lens=[50], pending_waited_ms=[5.0], decode_tokens=[9, 19, 4],
            decode_elapsed_ms=[90.0, 380.0, 40.0], decode_mean_ctx=1000, u_k=50, v_k=50)
HAND_SLO = dict(ttft_norm_ms_per_tok=0.5, tpot_ms=20.0, w_max=4, v_min=16, percentile=0.9)


def test_evaluate_split_hand_derived(monkeypatch):
    """Split (u, v) = (50, 50), co-run factor 1.25, L = 32, l_k = 4:
    t_p = 300/3/50 x 1.25 = 2.5 ms; rem = 2.5 x 28 = 70 ms (l.3).
    TTFT/SLO (l.4-7, R-18: SLO = 0.5 ms x input length):
      (70 + 10) / 50 = 1.6;  (70 + 20) / 100 = 0.9;
      pending 50 tok: own = 50/3/50 x 1.25 x 32 = 13.333 ms -> (5 + 70 + 13.333) / 25 = 3.5333.
    TPOT/SLO (l.8-10, R-14): iteration = 10/50 x 1.25 x 32 = 8 ms;
      (90 + 8)/10/20 = 0.49, (380 + 8)/20/20 = 0.97, (40 + 8)/5/20 = 0.48.
    Nearest-rank P90 of 3 = the largest; P50 = the 2nd smallest."""
    monkeypatch.setattr(PM, "layer_time", _stub_layer_time(1.25))
    P = PM.default_params(M=100)
    ttft, tpot, t_p = PM.evaluate_split(P, MODEL, dict(HAND), HAND_SLO, 50, 50)
    assert math.isclose(t_p, 2.5) and math.isclose(ttft, 3.5333333333333333) and math.isclose(tpot, 0.97)
    ttft, tpot, _ = PM.evaluate_split(P, MODEL, dict(HAND), dict(HAND_SLO, percentile=0.5), 50, 50)
    assert math.isclose(ttft, 1.6) and math.isclose(tpot, 0.49)


def test_evaluate_split_decode_pause_hand_derived(monkeypatch):
    """Decode pause (u, v) = (100, 0), v_k = 40: no co-runner, so
    t_p = 300/3/100 = 1 ms, rem = 28 ms; TTFT/SLO = 38/50 = 0.76, 48/100 = 0.48,
    pending (5 + 28 + 50/3/100 x 32) / 25 = 1.5333; the decodes wait one
    prefill layer and then run an iteration alone on v_k SMs:
    1 + 10/40 x 32 = 9 ms -> (90 + 9)/10/20 = 0.495, (380 + 9)/20/20 = 0.9725,
    (40 + 9)/5/20 = 0.49."""
    monkeypatch.setattr(PM, "layer_time", _stub_layer_time(1.25))
    P = PM.default_params(M=100)
    ttft, tpot, t_p = PM.evaluate_split(P, MODEL, dict(HAND, u_k=60, v_k=40), HAND_SLO, 100, 0)
    assert math.isclose(t_p, 1.0) and math.isclose(ttft, 1.5333333333333333) and math.isclose(tpot, 0.9725)


def _hand_state():
    return dict(HAND, pending_lens=[], pending_waited_ms=[])


HAND_SLO_LOOSE = dict(HAND_SLO, ttft_norm_ms_per_tok=100.0, tpot_ms=1e4)


def test_reduce_decode_hand_derived(monkeypatch):
    """Objective 0, both SLOs met everywhere: ReduceDecodeSM -> v = v_min = 16,
    u = 84; k = round(t_p / t_d) = round((100/84 x 1.25) / (10/16 x 1.25))
    = round(1.905) = 2."""
    monkeypatch.setattr(PM, "layer_time", _stub_layer_time(1.25))
    assert PM.choose_split(PM.default_params(M=100), MODEL, _hand_state(), HAND_SLO_LOOSE) == (84, 2)


def test_max_throughput_and_timesliced_hand_derived(monkeypatch):
    """Objective 1 (R-21 / R-22), n_pre = 300 tokens, 3 decodes.
    Time-sliced cycle: t_p = 1 ms, t_d = 0.1 ms alone on 100 SMs, k_ts = 10,
    cycle 2 ms -> (300 + 30) / 2 = 165 tokens/ms.
    Co-run, f = 1.25: t_p = 125/(100 - v), t_d = 12.5/v, k = round(t_p/t_d):
      v = 16: 1.488 / 0.781 -> k 2, cycle 1.5625, 306/1.5625 = 195.8
      v = 18: 1.524 / 0.694 -> k 2, cycle 1.5244, 306/1.5244 = 200.7  (best)
      v = 20: 1.5625 / 0.625 -> k 3, cycle 1.875, 309/1.875 = 164.8
      v = 22: 1.603 / 0.568 -> k 3, cycle 1.705, 181.3;  v = 24: k 3, 1.645, 187.9
    and t_p grows with v from there (v = 50: k 10, 330/2.5 = 132) -> (82, 2),
    since 200.7 > 165.  With f = 2 every co-run time doubles (v = 18:
    306/3.049 = 100.4 < 165) -> the time-sliced cycle (100, 10)."""
    P = PM.default_params(M=100)
    slo = dict(HAND_SLO_LOOSE, objective=1)
    monkeypatch.setattr(PM, "layer_time", _stub_layer_time(1.25))
    assert PM.choose_split(P, MODEL, _hand_state(), slo) == (82, 2)
    monkeypatch.setattr(PM, "layer_time", _stub_layer_time(2.0))
    assert PM.choose_split(P, MODEL, _hand_state(), slo) == (100, 10)


def _stub_saturating(f):
    """Decode that saturates HBM from 40 SMs on (the non-linearity co-running
    exploits, §8d feasibility): decode layer = 0.1 x max(1, 40 / m) ms, prefill
    layer = n / 3 / m ms, both x f under co-location."""
    def lt(shape, P, m, corun_m):
        if m <= 0:
            return math.inf
        g = f if corun_m > 0 else 1.0
        q = shape["q_lens"]
        ms = 0.1 * max(1.0, 40.0 / m) * g if all(x == 1 for x in q) else sum(q) / 3.0 / m * g
        return ms / 1e3
    return lt


def test_max_gain_hand_derived(monkeypatch):
    """R-23 (objective 2), M = 100, 300 prefill tokens, f = 1.25.  Alone on
    all SMs: t_p(N) = 1 ms, t_d(N) = 0.1 ms.  At decode SMs v:
    t_p = 125/(100 - v), t_d = 0.125 max(1, 40/v), gain(k) = (1 + 0.1k)/max(t_p, k t_d):
      v = 32: t_p 1.838,  r 11.76 -> k 11: 2.1/1.838 = 1.142;  k 12: 2.2/1.875 = 1.173
      v = 34: t_p 1.894,  r 12.88 -> k 12: 2.2/1.894 = 1.162;  k 13: 2.3/1.912 = 1.203
      v = 36: t_d 0.1389, r 14.06 -> k 14: 2.4/1.953 = 1.229;  k 15: 2.5/2.083 = 1.200
      v = 38: t_d 0.1316, r 15.32 -> k 15: 2.5/2.016 = 1.240;  k 16: 2.6/2.105 = 1.235
      v = 40: t_d 0.125,  r 16.67 -> k 16: 2.6/2.083 = 1.248;  k 17: 2.7/2.125 = 1.271  (best gain)
      v = 42: t_p 2.155,  r 17.24 -> k 17: 2.7/2.155 = 1.253;  k 18: 2.8/2.25 = 1.244
      v = 44: t_p 2.232,  r 17.86 -> k 17: 2.7/2.232 = 1.210;  k 18: 2.8/2.25 = 1.244
    (below 40 the decode is slower than linear, above it prefill loses SMs for
    nothing).  Best gain 1.271 at (u, k) = (60, 17); gains within 6 % of it
    (>= 1.1947: the model's resolution, its held-out MRE) are ties that go to
    the larger prefill share: v = 32 (1.173) is out, v = 34 is the
    smallest v in -> its larger gain, k = 13 -> (66, 13).  With f = 2 the best gain is
    2.7/3.4 = 0.79 < 1: co-running does not pay -> the time-sliced cycle
    (100, 10)."""
    P = PM.default_params(M=100)
    slo = dict(HAND_SLO_LOOSE, objective=2)
    monkeypatch.setattr(PM, "layer_time", _stub_saturating(1.25))
    assert PM.choose_split(P, MODEL, _hand_state(), slo) == (66, 13)
    monkeypatch.setattr(PM, "layer_time", _stub_saturating(2.0))
    assert PM.choose_split(P, MODEL, _hand_state(), slo) == (100, 10)
