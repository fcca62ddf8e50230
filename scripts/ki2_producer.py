"""KI2 follow-up: is the ~85 GB/s/SM ceiling of async copies (cp.async,
bulk) a property of the smem fill path?  Compare register-staged producers
(LDG.128 -> STS.128, mode 3) and plain LDG (mode 4) at 8 / 16 KB in flight
per warp (16 warps per SM) against cp.async (mode 2) and bulk (mode 1)."""
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
    for mode, param, name in ((3, 1, "ldg+sts 8KB/warp"), (3, 2, "ldg+sts 16KB/warp"), (4, 1, "ldg 8KB/warp"),
                              (4, 2, "ldg 16KB/warp"), (2, 0, "cp.async 192KB"), (1, 0, "bulk 192KB"),
                              (5, 1, "bulk 192KB + ldg 15 warps x 8KB")):
        for msm in (20, 40, 68, 100, 148):
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
