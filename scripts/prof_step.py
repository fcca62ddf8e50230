"""Run phase steps of the bench workload for ncu / timing (no JSON output).

  python scripts/prof_step.py --mode dec --p 108 --reps 3   # decode layer on sigma[108:N)
  python scripts/prof_step.py --mode pre --p 148            # prefill layer on all SMs
  python scripts/prof_step.py --mode corun --p 112 --k 4
Prints per-kernel event times (PROFILE flag) of the last rep.
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--mode", default="dec", choices=["dec", "pre", "corun", "timesliced"])
    ap.add_argument("--config", default="sharegpt-8b")
    ap.add_argument("--p", type=int, default=108)
    ap.add_argument("--k", type=int, default=1)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--quiet", action="store_true")
    ap.add_argument("--time", type=int, default=0, help="also time this many steps without PROFILE")
    ap.add_argument("--extra-flags", type=int, default=0, help="OR'ed into the step flags (e.g. 32 = UNFUSED_NORM)")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    S = bench.Step(a.config, max(1, a.k))
    B = S.B
    S.dec.layer_end = a.k
    flags = (B.TIMESLICED if a.mode == "timesliced" else B.CORUN) | a.extra_flags
    pre = a.mode in ("pre", "corun", "timesliced")
    dec = a.mode in ("dec", "corun", "timesliced")
    p = a.p if a.mode != "timesliced" else S.N
    for _ in range(a.reps - 1):
        S.enqueue(p, flags, pre, dec)
    torch.cuda.synchronize()
    if a.time:
        print(f"timed {S.time_steps(a.time, p, flags, pre, dec):.4f} ms/step over {a.time} steps")
    ms = S.time_steps(1, p, flags | B.PROFILE, pre, dec)
    if not a.quiet:
        print(f"step {ms:.4f} ms")
        for kind, ph, layer, t in S.bl.profile_read():
            print(f"  {'pre' if ph == 0 else 'dec'} L{layer} {kind:10s} {t:.4f} ms")


if __name__ == "__main__":
    main()
