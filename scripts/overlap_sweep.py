"""NEXT-4 experiment: co-run step with overlapping SM ranges (a shared band
of 2w SMs around the split p) vs the strict split, same work, interleaved
blocks.  python scripts/overlap_sweep.py --config sharegpt-8b --p 80 --k 7"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="sharegpt-8b")
    ap.add_argument("--p", type=int, default=80)
    ap.add_argument("--k", type=int, default=7)
    ap.add_argument("--bands", type=int, nargs="+", default=[0, 4, 8, 16, 24])
    a = ap.parse_args()
    torch.cuda.set_device(0)
    S = bench.Step(a.config, a.k)
    S.dec.layer_end = a.k
    B, N, p = S.B, S.N, a.p

    def t_ranges(w, n=5):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(S.sp)
        for _ in range(n):
            ev = torch.cuda.Event(); ev.record(S.sp); S.sd.wait_event(ev)
            S.bl.step_ranges(S.pre, S.dec, (0, min(N, p + w)), (max(0, p - w), N), B.CORUN, S.sp, S.sd)
            ev2 = torch.cuda.Event(); ev2.record(S.sd); S.sp.wait_event(ev2)
        e1.record(S.sp)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / n

    for _ in range(3):
        t_ranges(0)
    for w in a.bands:
        r = []
        for blk in range(6):
            if blk % 2 == 0:
                s0 = t_ranges(0); s1 = t_ranges(w)
            else:
                s1 = t_ranges(w); s0 = t_ranges(0)
            r.append(s0 / s1)
        print(json.dumps({"config": a.config, "p": p, "k": a.k, "band_half_width": w,
                          "speedup_vs_strict": float(np.median(r)), "ms_strict": s0, "ms_band": s1}), flush=True)


if __name__ == "__main__":
    main()
