"""Per-stage error diagnosis of one bf16 layer (op entry points vs oracle
diagnostics; test infrastructure, lives under tests/ with the other oracle
users).  Usage: python tests/tools/diag_layer.py [d H Hkv I prefill_len]"""
import sys, os
_T = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path[:0] = [os.path.dirname(_T), _T]
import numpy as np, torch
import oracle as O
from workload import synth
from harness import oracle_cfg, compare
import paper_conf_asplos_0001xc0l026_b200 as B

a = [int(x) for x in sys.argv[1:]] or [1024, 8, 2, 2816, 300]
m = synth.ModelShape("diag", a[0], a[1], a[2], 128, a[3], 1)
q_lens, ctx = [a[4]], [0]
lay = synth.paged_layout(q_lens, ctx, 16)
w = synth.layer_weights(m, 0)
pk, pv = synth.kv_pool(m, lay.n_blocks, 16, 0)
x = synth.hidden(a[4], m.d_model)
cfg = oracle_cfg(m)
wn = {k: (None if v is None else v.numpy()) for k, v in w.items()}
out_ref, dg = O.layer_forward(cfg, wn, pk.numpy().copy(), pv.numpy().copy(), q_lens, ctx, lay.block_table,
                              x.double().numpy(), diag=True)
bf = torch.bfloat16
pools = [(pk.to("cuda", bf).contiguous(), pv.to("cuda", bf).contiguous())]
bl = B.Bullet(B.Model.of(m), pools, 8192, 8192, 8192)
wg = {k: (None if v is None else v.to("cuda", bf)) for k, v in w.items()}
n, d, H, hd, I = a[4], m.d_model, m.n_heads, 128, m.d_ff
nq = (H + 2 * m.n_kv_heads) * hd
for kind in (1, 2, 4):
    pools[0][0].copy_(pk.to(bf)); pools[0][1].copy_(pv.to(bf))
    xg = x.cuda().contiguous()
    b = B.Batch(q_lens, ctx, lay.block_table, xg)
    h = torch.zeros(n, d, dtype=bf, device="cuda"); qkv = torch.zeros(n, nq, device="cuda")
    q = torch.zeros(n, H * hd, dtype=bf, device="cuda"); o = torch.zeros_like(q)
    act = torch.zeros(n, I, dtype=bf, device="cuda")
    bl.op_rmsnorm(xg, wg["g_attn"], h)
    bl.op_gemm(B.EPI_F32, h, wg["w_qkv"], qkv)
    if kind == 1:   # stage isolation: RMSNorm rounding flips, QKV GEMM accumulation error
        torch.cuda.synchronize()
        h_ref = O.round_bf16(O.rmsnorm(x.double().numpy(), w["g_attn"].double().numpy(), m.rms_eps))
        hg = h.float().cpu().numpy()
        ex = O.linear(hg.astype(np.float64), w["w_qkv"].double().numpy())
        f32 = torch.nn.functional.linear(torch.from_numpy(hg), w["w_qkv"].float()).numpy()
        gq = qkv.cpu().numpy()
        print(f"h flips {np.mean(hg != h_ref):.4f}   qkv GEMM vs fp64 (same h): gpu {compare(gq, ex)}  cpu-fp32 {compare(f32, ex)}")
    bl.op_rope_kv(b, 0, qkv, q)
    bl.op_attention(b, 0, q, o, kind=kind)
    bl.op_gemm(B.EPI_RESID, o, wg["w_o"], xg, resid=xg)
    bl.op_rmsnorm(xg, wg["g_mlp"], h)
    bl.op_gemm(B.EPI_SILU, h, wg["w_gate_up"], act, silu_half=I)
    bl.op_gemm(B.EPI_RESID, act, wg["w_down"], xg, resid=xg)
    torch.cuda.synchronize()
    qd = q.float().cpu().numpy(); od = o.float().cpu().numpy(); ad = act.float().cpu().numpy()
    print(f"kind={kind}  q flips {np.mean(qd != dg['q']):.4f}  o flips {np.mean(od != dg['o']):.4f} "
          f"o err {compare(od, dg['o'])}  a flips {np.mean(ad != dg['a']):.4f}  out {compare(xg.cpu().numpy(), out_ref)}"
          f"  delta {compare(xg.cpu().numpy() - x.numpy(), out_ref - x.double().numpy())}")
