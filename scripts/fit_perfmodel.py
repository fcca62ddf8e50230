"""Fit Bullet's performance-model parameters on the B200 (§3.2.2,
P:L147-149): isolated prefill and decode layer steps on a grid of SM counts
give the decay factors d_c(m), d_b(m); co-located runs give the contention
factors p_c, p_b.  Fits go through the product's own predictor (host-only
handle, `bullet_perf_create`), so the fitted JSON means exactly what
`bullet_model_predict` computes.  20 % of points are held out; the mean
relative error is reported beside the paper's 19.1 %.

    python scripts/fit_perfmodel.py [out.json]     (needs the GPU)
"""
import itertools
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
from workload import synth  # noqa: E402

M_GRID = [16, 32, 48, 64, 80, 96, 112, 128, 148]
PRE_SHAPES = [[512], [1024], [2048], [4096], [8192], synth.workload("sharegpt-8b").prefill_lens]
DEC_SHAPES = [[cl] * bs for bs in (32, 64, 128, 256) for cl in (512, 1024, 2048, 4096)] + \
    [list(synth.workload("sharegpt-8b").decode_ctx), list(synth.workload("arxiv-8b").decode_ctx)]
L_CO = 16
L_DEC = 4   # decode layer-steps per isolated decode point
# co-run points on the split grid the bench sweeps, with the bench's own
# request mixes (config 2: ShareGPT-shaped prompts x 128 decodes @ ~1k;
# config 3: 8k prompt x 256 decodes @ ~4k) plus two off-grid mixes
CORUN = [(pre, dec, p) for pre, dec in ((synth.workload("sharegpt-8b").prefill_lens, list(synth.workload("sharegpt-8b").decode_ctx)),
                                        ([8192], list(synth.workload("arxiv-8b").decode_ctx)),
                                        ([2048], [2048] * 256), ([4096], [512] * 64))
         for p in range(40, 140, 8)]


class Rig:
    def __init__(self):
        torch.cuda.set_device(0)
        self.m = synth.MODELS["llama3.1-8b"]
        w = synth.layer_weights(self.m, 0, device="cuda")
        self.w = {k: (None if v is None else v.bfloat16()) for k, v in w.items()}
        self.n_blocks = 256 * (6144 // 16 + 1) + 8192 // 16 + 64
        k, v = synth.kv_pool(self.m, self.n_blocks, 16, 0, device="cuda")
        self.pool = [(k.bfloat16(), v.bfloat16())]
        del k, v
        # L_CO layers sharing one weight set and one KV pool: a co-run point
        # runs k decode layer-steps against one prefill layer so the phases
        # overlap for the whole step (as in bullet_step), not just its start
        self.bl = B.Bullet(B.Model.of(self.m), self.pool * L_CO, 8192, 256, 8192 + 32)
        for l in range(L_CO):
            self.bl.set_layer_weights(l, self.w)
        self.N = self.bl.n_sms
        self.sp, self.sd = torch.cuda.Stream(), torch.cuda.Stream()

    def batch(self, q_lens, ctx_lens, first_block=0):
        """Block tables as the bench and a serving pool have them: a random
        permutation of the free blocks (fragmented KV — contiguous tables
        stream measurably faster and made round 2's first fit 30-50 %
        optimistic for KV-heavy decode batches)."""
        nb = [-(-(q + c) // 16) for q, c in zip(q_lens, ctx_lens)]
        total = sum(nb)
        rng = np.random.default_rng(first_block + 7)
        perm = first_block + rng.permutation(total).astype(np.int32)
        bt = np.zeros((len(nb), max(nb)), np.int32)
        pos = 0
        for i, n in enumerate(nb):
            bt[i, :n] = perm[pos:pos + n]
            pos += n
        pos += first_block
        x = torch.randn(sum(q_lens), self.m.d_model, device="cuda")
        torch.cuda.synchronize()   # x is read on the phase streams
        return B.Batch(q_lens, ctx_lens, bt, x, 0, 1), pos

    def time(self, pre, dec, p, reps=5):
        """Per-phase device times (ms) of one step; both phases start together."""
        for it in range(reps + 2):
            e0 = torch.cuda.Event(enable_timing=True)
            ep, ed = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(self.sp)
            self.sd.wait_event(e0)
            self.bl.step(pre, dec, p, B.CORUN, self.sp, self.sd)
            ep.record(self.sp)
            ed.record(self.sd)
            torch.cuda.synchronize()
            if it == 2:
                tp, td = [], []
            if it >= 2:
                tp.append(e0.elapsed_time(ep) if pre else 0.0)
                td.append(e0.elapsed_time(ed) if dec else 0.0)
        return float(np.median(tp)), float(np.median(td))


def measure():
    R = Rig()
    pts = []
    for lens in PRE_SHAPES:
        b, _ = R.batch(lens, [0] * len(lens))
        for m in M_GRID:
            tp, _ = R.time(b, None, m if m < R.N else R.N)
            pts.append({"kind": "pre", "q": lens, "c": [0] * len(lens), "m": m, "co": 0, "ms": tp})
    for ctx in DEC_SHAPES:
        bs = len(ctx)
        d, _ = R.batch([1] * bs, ctx, 0)
        d.layer_end = L_DEC   # per-layer time of a multi-layer decode step, as the co-run step runs it
        for m in M_GRID:
            _, td = R.time(None, d, R.N - m)
            pts.append({"kind": "dec", "q": [1] * bs, "c": list(ctx), "m": m, "co": 0, "ms": td / L_DEC})
    for lens, ctx, p in CORUN:
        bs = len(ctx)
        pre, used = R.batch(lens, [0] * len(lens))
        dec, _ = R.batch([1] * bs, ctx, used)
        tp0, _ = R.time(pre, None, p)                 # alone on the same SMs: the balance k
        _, td0 = R.time(None, dec, p)
        k = int(min(L_CO, max(1, round(tp0 / max(td0, 1e-6)))))
        dec.layer_end = k
        tp, td = R.time(pre, dec, p)
        pts.append({"kind": "pre", "q": lens, "c": [0] * len(lens), "m": p, "co": R.N - p, "ms": tp, "k": k})
        pts.append({"kind": "dec", "q": [1] * bs, "c": list(ctx), "m": R.N - p, "co": p, "ms": td / k, "k": k})
    return R.N, pts


def base_params(N):
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"bf16_tflops_sustained": 1395.1, "hbm_gbs": 6549.4}
    return {"M": N, "C_tflops": peaks.get("bf16_tflops_sustained", 1395.1), "B_gbs": peaks["hbm_gbs"],
            "d_c": {"m": [1, N], "v": [1.0, 1.0]}, "d_b": {"m": [1, N], "v": [1.0, 1.0]},
            "p_c": 1.0, "p_b": 1.0,
            "tiles": {"gemm_bm": 128, "gemm_bn": 256, "gemm_bk": 64, "min_k_blocks": 4, "attn_bq": 128,
                      "rows_per_unit": 8},
            "occ": {"gemm": 1, "attn": 2, "elem": 4}}


def predictor(m_shape, P, N):
    return B.PerfModel(B.Model.of(m_shape), N, json.dumps(P))


def fit(N, pts, m_shape):
    rng = np.random.default_rng(0)
    idx = rng.permutation(len(pts))
    held = set(idx[: len(pts) // 5].tolist())
    train = [p for i, p in enumerate(pts) if i not in held]
    test = [p for i, p in enumerate(pts) if i in held]
    P = base_params(N)
    grid = np.exp(np.linspace(np.log(0.05), np.log(3.0), 48))
    # per SM count m: the decode points fix the bandwidth decays of the GEMMs
    # and of the attention kernel (d_b, d_b_attn: the KV / weight byte mix
    # varies over the shapes), then the prefill points the compute decays
    # (d_c, d_c_attn) — R-12 / R-12b
    dc_v, db_v, dca_v, dba_v = [], [], [], []
    for m in M_GRID:
        def search(kind, keys, fixed):
            iso = [p for p in train if p["co"] == 0 and p["m"] == m and p["kind"] == kind]

            def err_of(x, y):
                Q = dict(P, **fixed, **{keys[0]: {"m": [1, N], "v": [x, x]}, keys[1]: {"m": [1, N], "v": [y, y]}})
                pm = predictor(m_shape, Q, N)
                e = sum((math.log(pm.predict_us(p["q"], p["c"], m, 0) / 1e3) - math.log(p["ms"])) ** 2 for p in iso)
                pm.close()
                return e
            best = min((err_of(x, y), x, y) for x, y in itertools.product(grid, grid))
            # refine: the coarse grid steps 9 %; search +-1 step at 0.5 % resolution
            step = grid[1] / grid[0]
            fine = lambda v: np.exp(np.linspace(np.log(v / step), np.log(v * step), 37))  # noqa: E731
            best = min([best] + [(err_of(x, y), x, y) for x, y in itertools.product(fine(best[1]), fine(best[2]))])
            return best[1], best[2]
        db, dba = search("dec", ("d_b", "d_b_attn"), {})
        fixed = {"d_b": {"m": [1, N], "v": [db, db]}, "d_b_attn": {"m": [1, N], "v": [dba, dba]}}
        dc, dca = search("pre", ("d_c", "d_c_attn"), fixed)
        dc_v.append(dc); db_v.append(db); dca_v.append(dca); dba_v.append(dba)
    P["d_c"] = {"m": M_GRID, "v": [float(x) for x in dc_v]}
    P["d_b"] = {"m": M_GRID, "v": [float(x) for x in db_v]}
    P["d_c_attn"] = {"m": M_GRID, "v": [float(x) for x in dca_v]}
    P["d_b_attn"] = {"m": M_GRID, "v": [float(x) for x in dba_v]}
    # co-location factors as functions of the phase's own SM count (R-12):
    # prefill co-run points fit p_c(m) (compute-bound kernels), decode ones
    # p_b(m) (bandwidth-bound), each grid point from the points nearest to it
    co = [p for p in train if p["co"] > 0]
    fgrid = np.linspace(0.4, 1.3, 181)

    def fit_table(kind, key):
        pts_k = [p for p in co if p["kind"] == kind]
        ms = sorted({p["m"] for p in pts_k})
        if not ms:
            return 1.0
        gm = [m for m in M_GRID if ms[0] - 16 <= m <= ms[-1] + 16] or [M_GRID[0], M_GRID[-1]]
        vals = []
        for g in gm:
            near = [p for p in pts_k if abs(p["m"] - g) <= 12] or \
                [min(pts_k, key=lambda p: abs(p["m"] - g))]
            best = (math.inf, 1.0)
            for f in fgrid:
                Q = dict(P, **{key: float(f)})
                pm = predictor(m_shape, Q, N)
                err = sum((math.log(pm.predict_us(p["q"], p["c"], p["m"], p["co"]) / 1e3) - math.log(p["ms"])) ** 2
                          for p in near)
                pm.close()
                if err < best[0]:
                    best = (err, float(f))
            vals.append(best[1])
        return {"m": [float(m) for m in gm], "v": vals}
    P["p_c"] = fit_table("pre", "p_c")
    P["p_b"] = fit_table("dec", "p_b")
    pm = predictor(m_shape, P, N)

    def mre(ps):
        return float(np.mean([abs(pm.predict_us(p["q"], p["c"], p["m"], p["co"]) / 1e3 - p["ms"]) / p["ms"] for p in ps]))
    P["fit"] = {"n_points": len(pts), "n_train": len(train), "n_heldout": len(test),
                "mre_train": mre(train), "mre_heldout": mre(test), "paper_mre": 0.191,
                "slo_accuracy_heldout": slo_accuracy(pm, test), "paper_slo_accuracy": 0.88,
                "source": "scripts/fit_perfmodel.py on B200"}
    return P


def split_heldout(pts):
    rng = np.random.default_rng(0)     # the same split fit() uses
    idx = rng.permutation(len(pts))
    held = set(idx[: len(pts) // 5].tolist())
    return [p for i, p in enumerate(pts) if i not in held], [p for i, p in enumerate(pts) if i in held]


def slo_accuracy(pm, pts, quantiles=(0.25, 0.5, 0.75)):
    """P:L311's second number: how often the model classifies a layer step
    the same way as the measurement with respect to a latency target ("meets"
    = time <= target).  Reading: targets at the 25 / 50 / 75 % quantiles of
    the measured times of each kind (prefill / decode layer steps), i.e. the
    decisions the scheduler takes near its SLO boundaries; mean over kinds
    and quantiles."""
    acc = []
    for kind in sorted({p["kind"] for p in pts}):
        ps = [p for p in pts if p["kind"] == kind]
        meas = np.array([p["ms"] for p in ps])
        pred = np.array([pm.predict_us(p["q"], p["c"], p["m"], p["co"]) / 1e3 for p in ps])
        for qn in quantiles:
            thr = float(np.quantile(meas, qn))
            acc.append(float(np.mean((pred <= thr) == (meas <= thr))))
    return float(np.mean(acc))


def evaluate(params_path, points_path):
    """Held-out MRE and SLO-classification accuracy of committed parameters
    (host-only model: no GPU)."""
    P = json.load(open(params_path))
    pts = json.load(open(points_path))
    _, test = split_heldout(pts)
    pm = predictor(synth.MODELS["llama3.1-8b"], P, P["M"])
    mre = float(np.mean([abs(pm.predict_us(p["q"], p["c"], p["m"], p["co"]) / 1e3 - p["ms"]) / p["ms"] for p in test]))
    return {"n_heldout": len(test), "mre_heldout": mre, "slo_accuracy_heldout": slo_accuracy(pm, test),
            "slo_accuracy_all": slo_accuracy(pm, pts), "paper": {"mre": 0.191, "slo_accuracy": 0.88}}


def main():
    if len(sys.argv) > 1 and sys.argv[1] == "--evaluate":
        pp = os.path.join(ROOT, "profiles", "perf_params_b200.json")
        print(json.dumps(evaluate(pp, pp.replace(".json", "_points.json"))))
        return
    if len(sys.argv) > 2 and sys.argv[1] == "--refit":   # fit again from saved points (host only)
        pts = json.load(open(sys.argv[2]))
        out = sys.argv[3] if len(sys.argv) > 3 else sys.argv[2].replace("_points.json", ".json")
        P = fit(148, pts, synth.MODELS["llama3.1-8b"])
        P["fit"]["points"] = os.path.basename(sys.argv[2])
        json.dump(P, open(out, "w"), indent=1)
        print(json.dumps(P["fit"]))
        return
    out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "perf_params_b200.json")
    t0 = time.time()
    N, pts = measure()
    P = fit(N, pts, synth.MODELS["llama3.1-8b"])
    P["fit"]["seconds"] = time.time() - t0
    json.dump(P, open(out, "w"), indent=1)
    json.dump(pts, open(out.replace(".json", "_points.json"), "w"))
    print(json.dumps(P["fit"]))


if __name__ == "__main__":
    main()
