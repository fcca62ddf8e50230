"""Decode-attention microbenchmark: bullet_op_attention on the bench
workload's decode batch (random KV, the bench's block tables) on the last
m SMs; prints KV GB/s and GB/s per SM.  Env:
BULLET_DEC_GROUPS (consumer groups per SM).

  python scripts/attn_dec_bench.py --config arxiv-8b --kind 3 --sms 60 148
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
    ap.add_argument("--config", default="sharegpt-8b")
    ap.add_argument("--kind", type=int, default=5)
    ap.add_argument("--sms", type=int, nargs="+", default=[60, 68, 148])
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--tag", default="")
    ap.add_argument("--uniform", type=int, nargs="*", default=None,
                    help="uniform contexts instead of the workload's: ctx values, n = 512K tokens / ctx")
    a = ap.parse_args()
    torch.cuda.set_device(0)
    wl = synth.workload(a.config)
    m = synth.MODELS[wl.model]
    for ctx in ([list(wl.decode_ctx)] if a.uniform is None else [[c] * max(1, (1 << 19) // c) for c in a.uniform]):
        run(a, m, ctx)


def run(a, m, ctx):
    n = len(ctx)
    lay = synth.paged_layout([1] * n, ctx, 16)
    torch.manual_seed(0)
    pk = torch.randn(lay.n_blocks, m.n_kv_heads, 16, m.head_dim, device="cuda").to(torch.bfloat16)
    pv = torch.randn_like(pk)
    bl = B.Bullet(B.Model.of(m), [(pk, pv)], n, n, max(ctx) + 32)
    q = torch.randn(n, m.n_heads * m.head_dim, device="cuda").to(torch.bfloat16)
    o = torch.empty_like(q)
    b = B.Batch([1] * n, ctx, lay.block_table, torch.zeros(n, m.d_model, device="cuda"))
    kv_bytes = sum(c + 1 for c in ctx) * m.n_kv_heads * m.head_dim * 2 * 2
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
        gbs = kv_bytes / us / 1e3
        sha = hashlib.sha256(o.view(torch.int16).cpu().numpy().tobytes()).hexdigest()[:16]   # A/B bit identity
        print(json.dumps({"sha": sha, "config": a.config, "kind": a.kind, "tag": a.tag, "ctx": ctx[0] if a.uniform else "mix",
                          "n": n, "units": n * m.n_kv_heads, "sms": msm, "us": round(us, 1),
                          "gbs": round(gbs), "gbs_per_sm": round(gbs / msm, 1)}), flush=True)


if __name__ == "__main__":
    main()
