"""Fused peer-memory all-reduce (PEER mode, NEXT-2) cost on ONE B200: the tp
ranks of a TP config are simulated as tp handles on disjoint halves/quarters
of the SMs (peer regions = local HBM, not NVLink).  For one phase at a time it
times a layer step of all ranks together (a) in PEER mode (GEMM partials +
fused reduce over the ranks' symmetric buffers) and (b) with tp_size = 1
handles of the same shard shapes (same kernels, same SM ranges, no
collective), so (a) - (b) is what the fused all-reduce adds.  Prints JSON
lines; numbers are local-memory stand-ins for NVLink, reported as such.

  python scripts/tp_sim_bench.py --config qwen14b-tp2 --reps 10
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_asplos_0001xc0l026_b200 as B  # noqa: E402
from paper_conf_asplos_0001xc0l026_b200 import parallel  # noqa: E402
from workload import synth  # noqa: E402


def build(wl, tp, peer, n_pre_tok, n_dec, maxpos, lay):
    m_full = synth.MODELS[wl.model]
    lm = B.Model.of(m_full.shard(tp))
    w = synth.layer_weights(m_full, 0, device="cuda")
    w = {k: (None if v is None else v.to(torch.bfloat16)) for k, v in w.items()}
    ranks = []
    for r in range(tp):
        ws = parallel.shard_layer_weights(w, B.Model.of(m_full), tp, r)
        k_, v_ = synth.kv_pool(m_full.shard(tp), lay.n_blocks, 16, 0, device="cuda")
        pools = [(k_.to(torch.bfloat16), v_.to(torch.bfloat16))]
        bl = B.Bullet(lm, pools, n_pre_tok, n_dec, maxpos, tp_size=tp if peer else 1, tp_rank=r if peer else 0)
        bl.set_layer_weights(0, ws)
        ranks.append(bl)
    if peer:
        bases = [bl.tp_base() for bl in ranks]
        for bl in ranks:
            bl.tp_connect(bases)
    return ranks


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="qwen14b-tp2")
    ap.add_argument("--reps", type=int, default=10)
    a = ap.parse_args()
    wl = synth.workload(a.config)
    tp = wl.tp
    q, c, n_pre = synth.combined_batch(wl)
    lay = synth.paged_layout(q, c, 16)
    n_p, n_d = sum(wl.prefill_lens), len(wl.decode_ctx)
    maxpos = max(x + y for x, y in zip(q, c)) + 16
    d = synth.MODELS[wl.model].d_model
    x_pre = synth.hidden(n_p, d, 0, device="cuda")
    x_dec = synth.hidden(n_d, d, 1, device="cuda")
    bt = lay.block_table
    for peer in (True, False):
        ranks = build(wl, tp, peer, n_p, n_d, maxpos, lay)
        N = ranks[0].n_sms
        g = (N // tp) & ~1
        for phase in ("prefill", "decode"):
            batches = []
            for bl in ranks:
                if phase == "prefill":
                    h = bl.tp_hidden(0, n_p) if peer else torch.empty_like(x_pre)
                    h.copy_(x_pre)
                    batches.append(B.Batch(wl.prefill_lens, [0] * n_pre, bt[:n_pre], h, 0, 1))
                else:
                    h = bl.tp_hidden(1, n_d) if peer else torch.empty_like(x_dec)
                    h.copy_(x_dec)
                    batches.append(B.Batch([1] * n_d, wl.decode_ctx, bt[n_pre:], h, 0, 1))
            streams = [torch.cuda.Stream() for _ in ranks]
            for s in streams:
                s.wait_stream(torch.cuda.current_stream())

            def step():
                for r, bl in enumerate(ranks):
                    rng = (r * g, (r + 1) * g)
                    if phase == "prefill":
                        bl.step_ranges(batches[r], None, rng, (0, 0), B.CORUN, streams[r], streams[r])
                    else:
                        bl.step_ranges(None, batches[r], (0, 0), rng, B.CORUN, streams[r], streams[r])
            for _ in range(3):
                step()
            torch.cuda.synchronize()
            ts = []
            for _ in range(a.reps):
                e0 = torch.cuda.Event(enable_timing=True)
                e0.record(streams[0])
                for s in streams[1:]:
                    s.wait_event(e0)
                step()
                e1 = torch.cuda.Event(enable_timing=True)
                for s in streams[1:]:
                    ev = torch.cuda.Event(); ev.record(s); streams[0].wait_event(ev)
                e1.record(streams[0])
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            for bl in ranks:
                bl.sync()
            n_tok = n_p if phase == "prefill" else n_d
            print(json.dumps({"config": a.config, "tp": tp, "phase": phase, "mode": "peer" if peer else "no-collective",
                              "sms_per_rank": g, "ms_per_layer": float(np.median(ts)), "tokens": n_tok,
                              "allreduce_bytes_per_rank_per_layer": 2 * 2 * (tp - 1) / tp * n_tok * d * 4}))
        for bl in ranks:
            bl.close()
        del ranks
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
