"""KI2b: per-SM HBM rate vs bytes in flight for LDG.128 and cp.async (40 SMs)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_asplos_0001xc0l026_b200 as B
from workload import synth
torch.cuda.set_device(0)
m = synth.ModelShape("ki2", 1024, 8, 2, 128, 2816, 1)
pools = [(torch.zeros(16, 2, 16, 128, dtype=torch.bfloat16, device="cuda"),) * 2]
bl = B.Bullet(B.Model.of(m), pools, 16, 16, 64)
buf = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
for msm in (20, 40, 60):
    for mode, param, inflight_kb in [(0, 2, 16), (0, 4, 32), (0, 8, 64), (0, 16, 128), (2, 2, 128), (2, 3, 192), (1, 0, 192)]:
        code = mode | (param << 8)
        bl.op_stream(buf, code, bl.n_sms - msm, bl.n_sms); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3):
            bl.op_stream(buf, code, bl.n_sms - msm, bl.n_sms)
        e1.record(); torch.cuda.synchronize()
        t = e0.elapsed_time(e1) / 3e3
        gbs = buf.numel() / t / 1e9 / msm
        print(json.dumps({"sms": msm, "mode": ["ldg", "bulk", "cp.async"][mode], "inflight_kb_per_sm": inflight_kb,
                          "gbs_per_sm": round(gbs, 1), "implied_latency_us": round(inflight_kb * 1024 / (gbs * 1e9) * 1e6, 2)}))
