"""NEXT-1: multi-step serving loop on the B200 (paper_conf_asplos_0001xc0l026_b200/serving.py).

Full Llama-3.1-8B (32 layers, random weights) serving a seeded Poisson trace
of ShareGPT-shaped requests; each scheduling cycle is one bullet_step (the
prefill batch advances one layer, the decode batch k layer-steps).  The same
trace is served under each policy and one JSON line per policy is printed:
TTFT / normalized TTFT / TPOT percentiles, SLO attainment (Table 2 ShareGPT
SLOs) and goodput, on virtual time = summed device time.

  python scripts/serve.py --rate 60 --duration 10 --policies bullet timesliced prefill_first chunked
"""
import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_asplos_0001xc0l026_b200 as B  # noqa: E402
from paper_conf_asplos_0001xc0l026_b200 import serving as SV  # noqa: E402
from workload import synth  # noqa: E402


class GpuStep:
    """One cycle = one bullet_step on two streams, device-timed."""

    def __init__(self, m, n_layers, n_blocks, max_prefill, max_decodes, perf_json):
        self.m = m
        self.pools = [(torch.zeros(n_blocks, m.n_kv_heads, 16, m.head_dim, dtype=torch.bfloat16, device="cuda"),
                       torch.zeros(n_blocks, m.n_kv_heads, 16, m.head_dim, dtype=torch.bfloat16, device="cuda"))
                      for _ in range(n_layers)]
        self.bl = B.Bullet(B.Model.of(m), self.pools, max_prefill, max_decodes, 4096,
                           perf_params_json=perf_json)
        for l in range(n_layers):
            w = synth.layer_weights(m, l, device="cuda")
            self.bl.set_layer_weights(l, {k: (None if v is None else v.bfloat16()) for k, v in w.items()})
        torch.cuda.synchronize()
        self.N = self.bl.n_sms
        self.sp, self.sd = torch.cuda.Stream(), torch.cuda.Stream()
        self.pre_id = self.dec_id = -1
        self.pre = self.dec = None
        self.rec = []   # per cycle (for --log-cycles): split, shapes, device ms

    @staticmethod
    def _table(reqs):
        w = max(len(r.blocks) for r in reqs)
        bt = np.zeros((len(reqs), w), np.int32)
        for i, r in enumerate(reqs):
            bt[i, :len(r.blocks)] = r.blocks
        return bt

    def __call__(self, pw, dw, p, mode):
        d = self.m.d_model
        if pw is not None:
            if pw.batch_id != self.pre_id:
                x = torch.randn(sum(pw.q_lens), d, device="cuda")
                self.pre = B.Batch(pw.q_lens, pw.ctx_lens, self._table(pw.reqs), x)
                self.pre_id = pw.batch_id
            self.pre.layer_begin, self.pre.layer_end = pw.layer_begin, pw.layer_end
        if dw is not None:
            if dw.batch_id != self.dec_id:   # new iteration: new token embeddings (synthetic)
                x = torch.randn(len(dw.q_lens), d, device="cuda")
                self.dec = B.Batch(dw.q_lens, dw.ctx_lens, self._table(dw.reqs), x)
                self.dec_id = dw.batch_id
            self.dec.layer_begin, self.dec.layer_end = dw.layer_begin, dw.layer_end
        cur = torch.cuda.current_stream()
        self.sp.wait_stream(cur)
        self.sd.wait_stream(cur)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(self.sp)
        self.sd.wait_event(e0)
        flags = B.TIMESLICED if mode == "timesliced" else B.CORUN
        self.bl.step(self.pre if pw is not None else None, self.dec if dw is not None else None, p, flags,
                     self.sp, self.sd)
        ej = torch.cuda.Event()
        ej.record(self.sd)
        self.sp.wait_event(ej)
        e1.record(self.sp)
        cur.wait_stream(self.sp)
        e1.synchronize()
        ms = e0.elapsed_time(e1)
        self.rec.append({"p": p, "mode": mode, "q": list(pw.q_lens) if pw is not None else [],
                         "pl": (pw.layer_end - pw.layer_begin) if pw is not None else 0,
                         "k": (dw.layer_end - dw.layer_begin) if dw is not None else 0,
                         "ctx": list(dw.ctx_lens) if dw is not None else [], "ms": ms})
        return ms


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rate", type=float, default=60.0, help="requests / s (Poisson)")
    ap.add_argument("--duration", type=float, default=10.0, help="seconds of arrivals")
    ap.add_argument("--layers", type=int, default=32)
    ap.add_argument("--policies", nargs="+", default=["bullet", "bullet_tput", "bullet_gain", "timesliced", "prefill_first",
                                                       "chunked"])
    ap.add_argument("--chunk-tokens", type=int, default=2048, help="chunked policy: token budget per iteration")
    ap.add_argument("--max-decodes", type=int, default=256)
    ap.add_argument("--max-prefill", type=int, default=8192)
    ap.add_argument("--blocks", type=int, default=24000)
    ap.add_argument("--static", type=int, nargs=2, default=[88, 6], help="policy static: prefill SMs, decode steps")
    ap.add_argument("--no-feedback", action="store_true", help="bullet policies: no online estimator feedback")
    ap.add_argument("--log-cycles", default=None, help="write every cycle (split, shapes, ms) as JSON lines here")
    ap.add_argument("--k-ts", type=int, default=0, help="decode layer-steps per cycle when time-sliced (0: model)")
    ap.add_argument("--seed", type=int, default=0)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    m = synth.MODELS["llama3.1-8b"]
    pj = os.path.join(ROOT, "profiles", "perf_params_b200.json")
    perf_json = open(pj).read() if os.path.exists(pj) else None
    g = GpuStep(m, a.layers, a.blocks, a.max_prefill, a.max_decodes, perf_json)
    # time-sliced k: the model's full-GPU balance of one prefill layer of a
    # typical batch against one decode layer-step of a typical decode batch
    k_ts = a.k_ts or max(1, round(g.bl.predict_us([400] * 8, [0] * 8, g.N) /
                                  g.bl.predict_us([1] * 128, [600] * 128, g.N)))
    # online level calibration (bullet_set_phase_scale): a typical
    # prefill layer and decode layer-step timed alone on the full GPU against
    # the model's prediction, before any policy runs
    cal = {}
    if not a.no_feedback:
        meas = {}
        for name, q, c in (("pre", [400] * 8, [0] * 8), ("dec", [1] * 128, [600] * 128)):
            blocks = list(range(sum(-(-(x + y) // 16) for x, y in zip(q, c))))
            reqs, pos = [], 0
            for x, y in zip(q, c):
                n = -(-(x + y) // 16)
                reqs.append(SV.Request(len(reqs), 0.0, max(x, 2), 2, blocks[pos:pos + n]))
                pos += n
            pw = SV.PhaseWork(reqs, q, c, 0, 4, -10 - len(meas))
            ts = []
            for _ in range(4):
                ts.append(g(pw if name == "pre" else None, pw if name == "dec" else None,
                            g.N if name == "pre" else 0, "corun"))
            g.rec = []
            meas[name] = float(np.median(ts[1:])) / 4
        pre_s = meas["pre"] / (g.bl.predict_us([400] * 8, [0] * 8, g.N) / 1e3)
        dec_s = meas["dec"] / (g.bl.predict_us([1] * 128, [600] * 128, g.N) / 1e3)
        g.bl.set_phase_scale(pre_s, dec_s)
        cal = {"prefill_layer_ms": meas["pre"], "decode_layer_ms": meas["dec"], "phase_scale": [pre_s, dec_s]}
    base = g.bl.colocation()
    for pol in a.policies:
        trace = SV.poisson_trace(a.rate, a.duration, seed=a.seed)
        g.bl.set_colocation(*base)   # every policy starts from the fitted factors
        fb = g.bl if (pol.startswith("bullet") and not a.no_feedback) else None
        loop = SV.ServingLoop(a.layers, g.N, g, g.bl.choose_split, pol, SV.BlockAllocator(a.blocks),
                              max_prefill_tokens=a.max_prefill, max_decodes=a.max_decodes, k_full=k_ts,
                              chunk_tokens=a.chunk_tokens, feedback_model=fb, static_split=tuple(a.static))
        t0 = time.perf_counter()
        res = loop.run(trace)
        res["policy"] = pol
        res["estimator_feedback"] = None if fb is None else {"corun_ratio": loop.fb_ratio,
                                                             "p_c_p_b": list(g.bl.colocation())}
        res.update(rate_req_s=a.rate, arrivals_s=a.duration, layers=a.layers, k_timesliced=k_ts, calibration=cal,
                   wall_s=time.perf_counter() - t0, model="llama3.1-8b", data="synthetic Poisson trace")
        ps = [c[1] for c in loop.log if 0 < c[1] < g.N]
        res["mean_prefill_sms_when_corun"] = float(np.mean(ps)) if ps else None
        ks = [c[2] for c in loop.log if c[2] > 0]
        res["mean_decode_steps_per_cycle"] = float(np.mean(ks)) if ks else None
        print(json.dumps(res), flush=True)
        if a.log_cycles:
            with open(f"{a.log_cycles}.{pol}.jsonl", "w") as f:
                for r in g.rec:
                    f.write(json.dumps(r) + "\n")
        g.rec = []


if __name__ == "__main__":
    main()
