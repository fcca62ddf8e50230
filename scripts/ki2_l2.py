"""KI2 follow-up: per-SM read rate from an L2-RESIDENT buffer (32 MB, re-read)
by load path — does the ~85 GB/s/SM async-copy ceiling also hold for L2
hits (the GEMM A operand), or is it a DRAM-latency effect?"""
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
    buf = torch.empty(2 << 30, dtype=torch.uint8, device="cuda")   # 2 GiB streamed per launch
    for mb in (32, 2048):
        for mode, param, name in ((1, 0, "bulk 192KB"), (2, 0, "cp.async 192KB"), (4, 1, "ldg 8KB/warp"),
                                  (5, 1, "bulk + ldg")):
            for msm in (20, 68, 148):
                lo = bl.n_sms - msm
                code = mode | (param << 8) | ((25 if mb == 32 else 0) << 16)   # 32 MB window: L2 hits
                reps = 3
                bl.op_stream(buf, code, lo, bl.n_sms)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                for _ in range(reps):
                    bl.op_stream(buf, code, lo, bl.n_sms)
                e1.record()
                torch.cuda.synchronize()
                t = e0.elapsed_time(e1) / reps * 1e-3
                print(json.dumps({"buffer_mb": mb, "mech": name, "sms": msm, "gbs": round(buf.numel() / t / 1e9, 1),
                                  "gbs_per_sm": round(buf.numel() / t / 1e9 / msm, 1)}), flush=True)


if __name__ == "__main__":
    main()
