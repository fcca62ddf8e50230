"""Per-CTA timeline of one phase step (bullet_trace_enable): for every traced
launch, when its CTAs entered, got their first operand stage, finished the
MMA issue / epilogue, and exited — and the gap to the previous launch.

  python scripts/trace_step.py --config sharegpt-8b --mode dec --p 80 --k 1
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_asplos_0001xc0l026_b200.bullet import KERNEL_KINDS  # noqa: E402


def analyse(rec, meta):
    rows, prev_end = [], None
    for i in range(len(meta)):
        r = rec[i]
        ok = r[:, 1] > 0
        if not ok.any():
            rows.append({"i": i, "kind": KERNEL_KINDS[meta[i][0]], "ctas": 0})
            continue
        r = r[ok].astype(np.int64)
        t0 = r[:, 1].min()
        us = lambda x: round(float(x) / 1e3, 2)  # noqa: E731
        row = {"i": i, "kind": KERNEL_KINDS[meta[i][0]], "phase": int(meta[i][1]), "layer": int(meta[i][2]),
               "ctas": int(ok.sum()), "span_us": us(r[:, 5].max() - t0),
               "entry_spread_us": us(np.percentile(r[:, 1], 90) - t0),
               "gap_from_prev_us": us(t0 - prev_end) if prev_end is not None else None}
        if (r[:, 2] > 0).any():
            g = r[r[:, 2] > 0]
            row["first_stage_us_med"] = us(np.median(g[:, 2] - g[:, 1]))
            row["mma_done_us_med"] = us(np.median(g[:, 3] - t0))
            row["mma_done_us_max"] = us(g[:, 3].max() - t0)
            row["epi_done_us_max"] = us(g[:, 4].max() - t0)
            if (g[:, 15] > 0).any():   # last accumulator ready (the MMAs of the CTA's last unit complete)
                row["acc_ready_us_med"] = us(np.median(g[g[:, 15] > 0][:, 15] - t0))
                row["acc_ready_us_max"] = us(g[:, 15].max() - t0)
            row["exit_us_med"] = us(np.median(g[:, 5] - t0))
            row["units_per_cta"] = [int(g[:, 6].min()), int(g[:, 6].max())]
        if (r[:, 7] > 0).any():
            row["partial_stored_us_max"] = us(r[r[:, 7] > 0][:, 7].max() - t0)
        if (r[:, 8] > 0).any():
            f = r[r[:, 8] > 0]
            row["fixup_ctas"] = int(len(f))
            row["fixups"] = int(f[:, 10].sum())
            row["fixup_start_us"] = [us(f[:, 8].min() - t0), us(f[:, 8].max() - t0)]
            row["fixup_end_us_max"] = us(f[:, 9].max() - t0)
            row["fixup_dur_us_med"] = us(np.median(f[:, 9] - f[:, 8]))
            g2 = f[f[:, 11] > 0]
            if len(g2):   # first item of group 0: start -> tile ready -> summed + stored -> signalled
                row["item_wait_us_med"] = us(np.median(g2[:, 12] - g2[:, 11]))
                row["item_ready_us_med"] = us(np.median(g2[:, 12] - t0))
                row["item_sum_store_us_med"] = us(np.median(g2[:, 13] - g2[:, 12]))
                row["item_signal_us_med"] = us(np.median(g2[:, 14] - g2[:, 13]))
        prev_end = r[:, 5].max() if (r[:, 5] > 0).any() else None
        rows.append(row)
    return rows


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="sharegpt-8b")
    ap.add_argument("--mode", default="dec", choices=["dec", "pre", "corun"])
    ap.add_argument("--p", type=int, default=80)
    ap.add_argument("--k", type=int, default=1)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    S = bench.Step(a.config, max(1, a.k))
    B = S.B
    S.dec.layer_end = a.k
    pre, dec = a.mode in ("pre", "corun"), a.mode in ("dec", "corun")
    for _ in range(3):
        S.enqueue(a.p, B.CORUN, pre, dec)
    torch.cuda.synchronize()
    ms = S.time_steps(3, a.p, B.CORUN, pre, dec)
    S.bl.trace_enable(64)
    S.enqueue(a.p, B.CORUN, pre, dec)
    torch.cuda.synchronize()
    rec, meta = S.bl.trace_read(64)
    S.bl.trace_enable(0)
    print(json.dumps({"config": a.config, "mode": a.mode, "p": a.p, "k": a.k, "step_ms": ms}))
    for row in analyse(rec, meta):
        print(json.dumps(row))


if __name__ == "__main__":
    main()
