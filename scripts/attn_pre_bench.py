"""Prefill-attention microbenchmark: bullet_op_attention (kind 4, the tcgen05
prefill kernel) on the workload's prompts (random Q / K / V in the paged
pool) on the last m SMs; prints causal TFLOP/s, the fraction of the measured
bf16 peak scaled to the m SMs, and a hash of the output (A/B bit identity).

  python scripts/attn_pre_bench.py --config arxiv-8b --sms 84 148
"""
import argparse
import hashlib
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_asplos_0001xc0l026_b200 as B  # noqa: E402
from workload import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="arxiv-8b")
    ap.add_argument("--kind", type=int, default=4)
    ap.add_argument("--sms", type=int, nargs="+", default=[84, 148])
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--tag", default="")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    wl = synth.workload(a.config)
    m = synth.MODELS[wl.model]
    lens = list(wl.prefill_lens)
    n = len(lens)
    lay = synth.paged_layout(lens, [0] * n, 16)
    torch.manual_seed(0)
    pk = torch.randn(lay.n_blocks, m.n_kv_heads, 16, m.head_dim, device="cuda").to(torch.bfloat16)
    pv = torch.randn_like(pk)
    T = sum(lens)
    bl = B.Bullet(B.Model.of(m), [(pk, pv)], T, n, max(lens) + 32)
    q = torch.randn(T, m.n_heads * m.head_dim, device="cuda").to(torch.bfloat16)
    o = torch.empty_like(q)
    b = B.Batch(lens, [0] * n, lay.block_table, torch.zeros(T, m.d_model, device="cuda"))
    # causal: query i attends to i + 1 keys; QK and PV 2 flops per MAC each
    flops = sum(L * (L + 1) // 2 for L in lens) * m.n_heads * m.head_dim * 4
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    for msm in a.sms:
        lo = bl.n_sms - msm
        for _ in range(3):
            bl.op_attention(b, 0, q, o, kind=a.kind, lo=lo)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.reps):
            bl.op_attention(b, 0, q, o, kind=a.kind, lo=lo)
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) / a.reps * 1e3
        tf = flops / us / 1e6
        sha = hashlib.sha256(o.view(torch.int16).cpu().numpy().tobytes()).hexdigest()[:16]
        print(json.dumps({"sha": sha, "config": a.config, "kind": a.kind, "tag": a.tag, "sms": msm, "us": round(us, 1),
                          "tflops": round(tf, 1),
                          "frac_of_partition_peak": round(tf / (peaks["bf16_tflops"] * msm / bl.n_sms), 3)}), flush=True)


if __name__ == "__main__":
    main()
