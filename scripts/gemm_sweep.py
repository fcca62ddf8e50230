"""Decode-GEMM sweep: time bullet_op_gemm on SM partitions of several sizes
(weight-streaming shapes of the decode side), report weight GB/s and GB/s/SM.

  python scripts/gemm_sweep.py [--m 256] [--plans 256,1 128,4 ...]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_asplos_0001xc0l026_b200.bullet import Bullet, Model, EPI_F32, EPI_SILU  # noqa: E402
from workload import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--m", type=int, nargs="+", default=[128, 256])
    ap.add_argument("--sms", type=int, nargs="+", default=[28, 48, 148])
    ap.add_argument("--plans", nargs="*", default=[""])
    ap.add_argument("--reps", type=int, default=20)
    a = ap.parse_args()
    torch.cuda.set_device(0)
    m = synth.MODELS["llama3.1-8b"]
    pools = [(torch.zeros(4, m.n_kv_heads, 16, m.head_dim, dtype=torch.bfloat16, device="cuda"),
              torch.zeros(4, m.n_kv_heads, 16, m.head_dim, dtype=torch.bfloat16, device="cuda"))]
    mm = Model.of(m)
    B = Bullet(mm, pools, 512, 512, 8192)
    d, I = m.d_model, m.d_ff
    nq = (m.n_heads + 2 * m.n_kv_heads) * m.head_dim
    shapes = [("qkv", nq, d, EPI_F32), ("o_proj", d, m.n_heads * m.head_dim, EPI_F32),
              ("gate_up", 2 * I, d, EPI_SILU), ("down", d, I, EPI_F32)]
    st = torch.cuda.current_stream()
    for plan in a.plans:
        if plan:
            os.environ["BULLET_GEMM_PLAN"] = plan
        else:
            os.environ.pop("BULLET_GEMM_PLAN", None)
        for M in a.m:
            for name, N, K, epi in shapes:
                A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
                W = (torch.randn(N, K, device="cuda") * 0.02).to(torch.bfloat16)
                out = torch.empty(M, N // 2 if epi == EPI_SILU else N, device="cuda",
                                  dtype=torch.bfloat16 if epi == EPI_SILU else torch.float32)
                for n_sm in a.sms:
                    lo = B.n_sms - n_sm
                    for _ in range(3):
                        B.op_gemm(epi, A, W, out, silu_half=I if epi == EPI_SILU else 0, lo=lo)
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record(st)
                    for _ in range(a.reps):
                        B.op_gemm(epi, A, W, out, silu_half=I if epi == EPI_SILU else 0, lo=lo)
                    e1.record(st)
                    torch.cuda.synchronize()
                    us = e0.elapsed_time(e1) * 1e3 / a.reps
                    gbs = N * K * 2 / us / 1e3
                    print(f"plan={plan or 'auto':7s} M={M:4d} {name:8s} sms={n_sm:3d} {us:8.1f} us  "
                          f"{gbs:7.0f} GB/s  {gbs / n_sm:6.1f} GB/s/SM  {2 * M * N * K / us / 1e6:7.1f} TFLOP/s", flush=True)


if __name__ == "__main__":
    main()
