"""KI2: HBM read GB/s reachable from m SMs, per load mechanism (mode 0 LDG.128,
1 cp.async.bulk, 2 cp.async).  Prints one JSON line per (mode, m)."""
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
    buf = torch.empty(2 << 30, dtype=torch.uint8, device="cuda")   # 2 GiB >> L2
    ms_list = [int(x) for x in (sys.argv[1:] or [8, 16, 24, 32, 40, 48, 64, 80, 96, 112, 128, 148])]
    for mode in (0, 1, 2):
        for msm in ms_list:
            lo = bl.n_sms - msm
            bl.op_stream(buf, mode, lo, bl.n_sms)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            for _ in range(3):
                bl.op_stream(buf, mode, lo, bl.n_sms)
            e1.record()
            torch.cuda.synchronize()
            t = e0.elapsed_time(e1) / 3 * 1e-3
            print(json.dumps({"mode": mode, "sms": msm, "gbs": buf.numel() / t / 1e9,
                              "gbs_per_sm": buf.numel() / t / 1e9 / msm}))


if __name__ == "__main__":
    main()
