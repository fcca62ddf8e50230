"""Layer-step error vs the CPU oracle through the product path (bullet_step,
the kernels and GEMM plans the bench runs), for the R-4e precision readings.

  python scripts/precision_layer.py llama3.1-70b qwen2.5-14b [--pre 40,17] [--dec 33,1,200,64] [--sample 256]

Prints one JSON line per model: max-abs / mean-rel (normalized L1) of the
prefill and decode outputs.  Knobs (env): BULLET_GEMM_KCHUNK, _ONLY, _MODE.
Test infrastructure (imports the oracle): lives beside the other scripts
that compare against it and is never on the product path."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [ROOT, os.path.join(ROOT, "tests")]

import numpy as np  # noqa: E402
import torch  # noqa: E402

from harness import Setup, compare, phase_streams  # noqa: E402
from workload import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("models", nargs="+")
    ap.add_argument("--pre", default="40,17")
    ap.add_argument("--dec", default="33,1,200,64")
    ap.add_argument("--sample", type=int, default=0, help="row-sample the prefill rows (0 = all)")
    ap.add_argument("--p", type=int, default=74)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    pre = [int(x) for x in a.pre.split(",") if x]
    dec = [int(x) for x in a.dec.split(",") if x]
    for name in a.models:
        m = synth.MODELS[name]
        S = Setup(m, pre, dec, n_layers=1)
        mask = None
        if a.sample and sum(pre) > a.sample:
            rng = np.random.default_rng(7)
            mask = np.zeros(sum(pre), dtype=np.uint8)
            mask[rng.choice(sum(pre), a.sample, replace=False)] = 1
            mask[np.cumsum(pre) - 1] = 1      # every request's last row
        ref = S.oracle(row_mask_pre=mask)
        p_b, d_b = S.batches()
        S.bl.step(p_b, d_b, a.p, S.B.CORUN, *phase_streams())
        torch.cuda.synchronize()
        out = {"model": name, "pre": pre if len(pre) < 10 else f"{len(pre)} reqs / {sum(pre)} tok",
               "dec": len(dec), "kc": os.environ.get("BULLET_GEMM_KCHUNK"),
               "only": os.environ.get("BULLET_GEMM_KCHUNK_ONLY"), "mode": os.environ.get("BULLET_GEMM_KCHUNK_MODE")}
        g = p_b.hidden.cpu().numpy()
        if mask is not None:
            sel = mask.astype(bool)
            mx, mr = compare(g[sel], ref["pre"][sel])
        else:
            mx, mr = compare(g, ref["pre"])
        out["pre_maxabs"], out["pre_meanrel"] = mx, mr
        mx, mr = compare(d_b.hidden.cpu().numpy(), ref["dec"])
        out["dec_maxabs"], out["dec_meanrel"] = mx, mr
        print(json.dumps(out), flush=True)
        S.bl.close()
        del S
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
