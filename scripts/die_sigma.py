"""Die-aware sigma (SURVEY §8a SG): the same co-run step and
its phases alone with sigma in smid order, die-grouped and die-interleaved
(BULLET_SIGMA), plus the HBM stream rate of the decode range (KI2 kernel).

  python scripts/die_sigma.py --config sharegpt-8b --p 76 --k 8
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="sharegpt-8b")
    ap.add_argument("--p", type=int, default=76)
    ap.add_argument("--k", type=int, default=8)
    ap.add_argument("--reps", type=int, default=10)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    import bench
    for pol in ("sorted", "die", "interleave", "sorted"):
        os.environ["BULLET_SIGMA"] = pol
        S = bench.Step(a.config, a.k)
        B = S.B
        N = S.N
        S.dec.layer_end = a.k
        for _ in range(3):
            S.enqueue(a.p, B.CORUN)
        co = S.time_steps(a.reps, a.p, B.CORUN)
        pre = S.time_steps(a.reps, a.p, B.CORUN, dec=False)
        dec = S.time_steps(a.reps, a.p, B.CORUN, pre=False)
        buf = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        for _ in range(2):
            S.bl.op_stream(buf, mode=0, lo=a.p, hi=N)
        e0.record()
        for _ in range(5):
            S.bl.op_stream(buf, mode=0, lo=a.p, hi=N)
        e1.record()
        torch.cuda.synchronize()
        gbs = 5 * buf.numel() / (e0.elapsed_time(e1) * 1e-3) / 1e9
        dies = S.bl.sm_dies()
        print(json.dumps({"sigma": pol, "config": a.config, "p": a.p, "k": a.k, "corun_ms": co, "prefill_ms": pre,
                          "decode_ms": dec, "decode_range_stream_gbs": gbs, "fallbacks": S.bl.gate_fallbacks(),
                          "prefill_range_dies": [dies[:a.p].count(0), dies[:a.p].count(1)],
                          "decode_range_dies": [dies[a.p:].count(0), dies[a.p:].count(1)]}), flush=True)
        S.bl.close()
        del S, buf
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
