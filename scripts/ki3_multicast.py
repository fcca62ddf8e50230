"""KI3: per-SM delivered bandwidth of bulk copies with and without TMA
multicast (clusters of 2).  If multicast delivers more bytes
per SM than the ~85 GB/s/SM unicast ceiling, sharing the decode GEMMs'
activation tile across a CTA pair pays."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_0001xc0l026_b200 as B  # noqa: E402
from workload import synth  # noqa: E402


def main():
    torch.cuda.set_device(0)
    m = synth.ModelShape("ki3", 1024, 8, 2, 128, 2816, 1)
    pools = [(torch.zeros(16, 2, 16, 128, dtype=torch.bfloat16, device="cuda"),) * 2]
    bl = B.Bullet(B.Model.of(m), pools, 16, 16, 64)
    for window in (2 << 30, 32 << 20):   # DRAM stream, then an L2-resident 32 MB window
        buf = torch.empty(window, dtype=torch.uint8, device="cuda")
        reps = 3 if window > (1 << 30) else 60
        for n in (20, 40, 68, 148):
            for mc in (0, 1):
                bl.op_stream_mc(buf, mc, n)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                for _ in range(reps):
                    bl.op_stream_mc(buf, mc, n)
                e1.record()
                torch.cuda.synchronize()
                t = e0.elapsed_time(e1) / reps * 1e-3
                # every SM receives all bytes of its cluster's units: delivered = 2 x buffer / ... per SM
                delivered = 2 * buf.numel()          # both CTAs of a cluster receive each unit
                print(json.dumps({"window_mb": window >> 20, "ctas": n, "multicast": mc,
                                  "hbm_or_l2_gbs": round(buf.numel() / t / 1e9, 1),
                                  "delivered_gbs_per_sm": round(delivered / t / 1e9 / n, 1)}), flush=True)


if __name__ == "__main__":
    main()
