"""KI2 follow-up: is the ~85 GB/s/SM bulk-copy ceiling per issuing thread or
per SM?  mode 1 (bulk copies, one issuer, 6 x 32 KB ring) vs two CTAs per SM
each issuing from its own 3 x 32 KB ring (same bytes in flight per SM)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_0001xc0l026_b200 as B  # noqa: E402
from workload import synth  # noqa: E402


def main():
    torch.cuda.set_device(0)
    m = synth.ModelShape("ki2", 1024, 8, 2, 128, 2816, 1)
    pools = [(torch.zeros(16, 2, 16, 128, dtype=torch.bfloat16, device="cuda"),) * 2]
    bl = B.Bullet(B.Model.of(m), pools, 16, 16, 64)
    buf = torch.empty(2 << 30, dtype=torch.uint8, device="cuda")
    for mode, param, name in ((1, 0, "1 CTA/SM, 1 issuer x 6 stages"), (1, 3, "2 CTAs/SM, 1 issuer x 3 stages each"),
                              (7, 0, "1 CTA/SM, 2 issuer threads x 3 stages each"),
                              (8, 0, "1 CTA/SM, 1 issuer x 6 stages, one atomic per 8 units")):
        for msm in (20, 40, 68):
            lo = bl.n_sms - msm
            code = mode | (param << 8)
            bl.op_stream(buf, code, lo, bl.n_sms)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(3):
                bl.op_stream(buf, code, lo, bl.n_sms)
            e1.record()
            torch.cuda.synchronize()
            t = e0.elapsed_time(e1) / 3 * 1e-3
            print(json.dumps({"mech": name, "sms": msm, "gbs": round(buf.numel() / t / 1e9, 1),
                              "gbs_per_sm": round(buf.numel() / t / 1e9 / msm, 1)}), flush=True)


if __name__ == "__main__":
    main()
