"""Per-kind GEMM plan sweep on the decode side of the bench workload:
time the decode layer-step with BULLET_PROFILE for each forced plan
(BULLET_GEMM_PLAN_K<kind> = "mh,bn,sk") and print the GEMM's event time.

  python scripts/decode_gemm_plans.py --p 80 0
"""
import argparse
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402

KINDS = {"qkv": 2, "o_proj": 5, "gate_up": 7, "down": 8}
PLANS = {   # "mh,bn,sk": sk 1 streams the ragged remainder over K (stream-K + fixup phase)
    "qkv": ["", "1,256,0", "1,256,1", "1,128,0", "1,128,1"],
    "o_proj": ["", "1,64,0", "1,64,1", "1,128,0", "1,128,1", "1,256,1"],
    "gate_up": ["", "1,256,0", "1,256,1", "1,128,0", "1,128,1"],
    "down": ["", "1,128,0", "1,128,1", "1,256,1", "1,64,0"],
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="sharegpt-8b")
    ap.add_argument("--p", type=int, nargs="+", default=[80, 0])
    ap.add_argument("--k", type=int, default=4)
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    S = bench.Step(a.config, a.k)
    B = S.B
    S.dec.layer_end = a.k
    for p in a.p:
        for name, plans in PLANS.items():
            for plan in plans:
                key = f"BULLET_GEMM_PLAN_K{KINDS[name]}"
                if plan:
                    os.environ[key] = plan
                else:
                    os.environ.pop(key, None)
                for _ in range(2):
                    S.enqueue(p, B.CORUN, False, True)
                tot = defaultdict(float)
                step = S.time_steps(a.reps, p, B.CORUN, False, True)
                S.bl.profile_read()
                S.time_steps(a.reps, p, B.CORUN | B.PROFILE, False, True)
                for kind, ph, layer, t in S.bl.profile_read():
                    tot[kind] += t
                n = a.reps * a.k
                print(f"p={p:3d} {name:8s} plan={plan or 'auto':9s} {tot[name] / n * 1e3:7.1f} us   "
                      f"(step {step / a.k * 1e3:6.1f} us/layer)", flush=True)
            os.environ.pop(f"BULLET_GEMM_PLAN_K{KINDS[name]}", None)


if __name__ == "__main__":
    main()
