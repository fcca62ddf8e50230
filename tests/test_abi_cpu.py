"""CPU checks of the C-ABI library (no GPU): it loads, exports every symbol
include/bullet.h declares, and its host-side performance model / split
decision (C++) equal the oracle's plain reading (oracle/perfmodel.py)."""
import json

import numpy as np
import os

import pytest

import paper_conf_asplos_0001xc0l026_b200 as B
from oracle import perfmodel as PM


def test_library_exports_every_declared_symbol():
    L = B.lib()
    syms = B.declared_symbols()
    assert len(syms) >= 15
    missing = [s for s in syms if not hasattr(L, s)]
    assert not missing, missing


def test_library_is_sm100a_only():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", B.bullet._build.OUT],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", B.bullet._build.OUT],
                          capture_output=True, text=True).stdout
    for mnem in ("UTCHMMA", "UTMALDG", "LDTM"):   # tcgen05.mma, TMA, tcgen05.ld
        assert mnem in sass


MODELS = {
    "llama8b": dict(d=4096, H=32, Hkv=8, hd=128, I=14336, elt=2),
    "tiny": dict(d=256, H=4, Hkv=2, hd=64, I=768, elt=4),
}


def _pm(name, n_sms=148, params=None):
    m = MODELS[name]
    model = B.Model(m["d"], m["H"], m["Hkv"], m["hd"], m["I"], dtype="bf16" if m["elt"] == 2 else "fp32")
    return B.PerfModel(model, n_sms, json.dumps(params) if params else None)


def _fitted_params():
    P = PM.default_params()
    P["d_c"] = {"m": [8, 40, 100, 148], "v": [0.6, 0.8, 0.9, 0.85]}
    P["d_b"] = {"m": [8, 32, 148], "v": [1.9, 1.5, 0.9]}
    P["p_c"], P["p_b"] = 0.93, 0.81
    return P


@pytest.mark.parametrize("params", [None, "fitted"])
@pytest.mark.parametrize("name", ["llama8b", "tiny"])
def test_predict_equals_oracle_eq2(name, params):
    P = _fitted_params() if params else PM.default_params()
    pm = _pm(name, params=P)
    rng = np.random.default_rng(0)
    shape = dict(MODELS[name])
    cases = [([4096], [0]), ([512] * 8, [0] * 8), ([1] * 128, list(rng.integers(512, 1537, 128))),
             ([8192], [0]), ([33, 1, 1], [0, 5, 700]), ([1] * 3, [0, 0, 0])]
    for q, c in cases:
        for m, co in [(148, 0), (100, 48), (16, 132), (2, 0), (77, 71)]:
            got = pm.predict_us(q, c, m, co)
            ref = PM.layer_time(dict(shape, q_lens=list(q), ctx_lens=[int(x) for x in c]), P, m, co) * 1e6
            assert got == pytest.approx(ref, rel=1e-12), (q[:3], m, co)


def test_choose_split_equals_oracle_on_random_states():
    P = _fitted_params()
    pm = _pm("llama8b", params=P)
    model = MODELS["llama8b"]
    rng = np.random.default_rng(1)
    seen = set()
    for trial in range(120):
        n_pre = int(rng.integers(0, 3)); n_pend = int(rng.integers(0, 6)); n_dec = int(rng.integers(0, 40))
        st = dict(layers_done=int(rng.integers(0, 32)), total_layers=32,
                  prefill_lens=[int(x) for x in rng.integers(128, 8192, n_pre)],
                  prefill_waited_ms=[float(x) for x in rng.uniform(0, 3000, n_pre)],
                  pending_lens=[int(x) for x in rng.integers(64, 4096, n_pend)],
                  pending_waited_ms=[float(x) for x in rng.uniform(0, 2000, n_pend)],
                  decode_tokens=[int(x) for x in rng.integers(0, 300, n_dec)],
                  decode_elapsed_ms=[float(x) for x in rng.uniform(0, 40000, n_dec)],
                  decode_mean_ctx=float(rng.uniform(100, 4000)),
                  u_k=0, v_k=0)
        st["v_k"] = int(rng.integers(8, 140)); st["u_k"] = 148 - st["v_k"]
        slo = {"ttft_norm_ms_per_tok": float(rng.choice([3.0, 1.5, 0.3])),
               "tpot_ms": float(rng.choice([150.0, 200.0, 175.0, 30.0])),
               "w_max": int(rng.integers(0, 5)), "v_min": int(rng.choice([8, 16, 24])),
               "percentile": 0.9, "objective": int(trial % 3)}   # all objectives (R-21, R-23)
        ref = PM.choose_split(P, model, st, slo)
        got = pm.choose_split(st, slo)
        assert got == ref, (trial, got, ref)
        seen.add(ref[0])
    assert len(seen) >= 4   # several distinct decisions exercised


def test_host_only_handle_rejects_gpu_calls():
    pm = _pm("tiny")
    pm.sync()   # no-op on a host-only handle
    assert B.lib().bullet_step(pm.h, None, None, 0, 0, None, None) == -7
    assert B.lib().bullet_op_rmsnorm(pm.h, None, 0, None, None, 0, 1, None) == -7


def test_malformed_perf_params_rejected():
    with pytest.raises(B.BulletError) as e:
        _pm("tiny", params=None).__class__(B.Model(256, 4, 2, 64, 768), 148, "{\"d_c\": [1,2")
    assert e.value.code == -1


def test_predict_rejects_bad_sm_count():
    pm = _pm("llama8b")
    with pytest.raises(B.BulletError) as e:
        pm.predict_us([10], [0], 0)
    assert e.value.code == -4
    with pytest.raises(B.BulletError):
        pm.predict_us([10], [0], 149)


def test_fitted_perf_params_load_and_match_oracle():
    """profiles/perf_params_b200.json (fitted on the B200 by
    scripts/fit_perfmodel.py) parses in the C++ model and predicts exactly
    what the oracle's Eq. 2 reading predicts with the same parameters."""
    import os
    path = os.path.join(os.path.dirname(os.path.dirname(__file__)), "profiles", "perf_params_b200.json")
    if not os.path.exists(path):
        pytest.skip("no fitted parameters yet")
    P = json.load(open(path))
    pm = _pm("llama8b", params=P)
    shape = dict(MODELS["llama8b"])
    for q, c in [([4096], [0]), ([1] * 128, [1024] * 128), ([512] * 8, [0] * 8)]:
        for m, co in [(148, 0), (40, 108), (100, 48), (16, 0)]:
            got = pm.predict_us(q, c, m, co)
            ref = PM.layer_time(dict(shape, q_lens=q, ctx_lens=c), P, m, co) * 1e6
            assert got == pytest.approx(ref, rel=1e-12)
    assert P["fit"]["mre_heldout"] < 0.5


def test_header_is_plain_c99(tmp_path):
    """include/bullet.h is a C ABI: it must compile as strict C99 on its own
    (no C++ or torch types cross the boundary)."""
    import shutil
    import subprocess
    gcc = shutil.which("gcc")
    if gcc is None:
        pytest.skip("no gcc")
    src = tmp_path / "t.c"
    src.write_text('#include "bullet.h"\nint main(void) { bullet_handle *h = 0; (void)h; return 0; }\n')
    inc = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include")
    r = subprocess.run([gcc, "-std=c99", "-Wall", "-Wextra", "-pedantic", "-Werror", "-fsyntax-only", "-I", inc, str(src)],
                       capture_output=True, text=True)
    assert r.returncode == 0, r.stderr


def test_phase_scale_equals_oracle():
    """Online level calibration (bullet_set_phase_scale): prefill- and
    decode-shaped predictions scale by their own factor, as in the oracle."""
    P = _fitted_params()
    pm = _pm("llama8b", params=P)
    pm.set_phase_scale(1.3, 0.7)
    assert pm.phase_scale() == (1.3, 0.7)
    shape = dict(MODELS["llama8b"])
    Q = dict(P, scale_pre=1.3, scale_dec=0.7)
    for q, c in [([4096], [0]), ([1] * 64, [900] * 64), ([33, 1], [0, 5])]:
        for m, co in [(148, 0), (80, 68)]:
            ref = PM.layer_time(dict(shape, q_lens=q, ctx_lens=c), Q, m, co) * 1e6
            assert pm.predict_us(q, c, m, co) == pytest.approx(ref, rel=1e-12)
    with pytest.raises(Exception):
        pm.set_phase_scale(0.0, 1.0)
