"""NEXT-1 on the device: the serving loop (serving.py) drives bullet_step on
the B200 for ~20 scheduling cycles of a seeded Poisson trace, with Alg. 1
(bullet_choose_split) deciding every cycle, prefill batches advancing a
layer group per cycle and finished prompts joining the decode batch
copy-free (their block-table rows are kept).  Every layer each
phase runs in a cycle is checked against the CPU oracle, fed the device's own
input to that layer and the device's KV pool as the cached context (R-4c):
outputs within the north-star bar (prefill rows sampled, decode rows all) and
this layer's new k / v at exactly the slots the block table names, equal to
the oracle's up to one-step rounding flips.  The cycle's layers run as
single-layer co-run steps at the loop's split (a multi-layer step is bit-
identical to its single-layer steps: test_gpu_layer)."""
import numpy as np
import pytest
import torch

import oracle as O
from harness import compare, oracle_cfg
from workload import synth

pytestmark = pytest.mark.gpu

M = synth.ModelShape("serve-small", 1024, 8, 2, 128, 2816, 4)
N_BLOCKS = 3000


class CheckedStep:
    def __init__(self, B, bl, w_cpu, pools):
        self.B, self.bl, self.w_cpu, self.pools = B, bl, w_cpu, pools
        self.cfg = oracle_cfg(M)
        self.gen = torch.Generator(device="cuda").manual_seed(5)
        self.pre_id = self.dec_id = -1
        self.x_pre = self.x_dec = None
        self.checked = {"pre": 0, "dec": 0}
        self.worst = 0.0
        self.sp, self.sd = torch.cuda.Stream(), torch.cuda.Stream()

    @staticmethod
    def table(reqs):
        w = max(len(r.blocks) for r in reqs)
        bt = np.zeros((len(reqs), w), np.int32)
        for i, r in enumerate(reqs):
            bt[i, :len(r.blocks)] = r.blocks
        return bt

    def _oracle(self, layer, x, q, c, bt, pk, pv, mask=None):
        w = {k: (None if v is None else v.numpy()) for k, v in self.w_cpu[layer].items()}
        return O.layer_forward(self.cfg, w, pk, pv, q, c, bt, np.asarray(x, dtype=np.float64), row_mask=mask)

    def __call__(self, pw, dw, p, mode):
        B = self.B
        if pw is not None and pw.batch_id != self.pre_id:
            self.x_pre = torch.randn(sum(pw.q_lens), M.d_model, device="cuda", generator=self.gen)
            self.pre_id = pw.batch_id
        if dw is not None and dw.batch_id != self.dec_id:
            self.x_dec = torch.randn(len(dw.q_lens), M.d_model, device="cuda", generator=self.gen)
            self.dec_id = dw.batch_id
        n_p = (pw.layer_end - pw.layer_begin) if pw is not None else 0
        n_d = (dw.layer_end - dw.layer_begin) if dw is not None else 0
        flags = B.TIMESLICED if mode == "timesliced" else B.CORUN
        for i in range(max(n_p, n_d)):
            phases = []
            if i < n_p:
                phases.append(("pre", pw, pw.layer_begin + i, self.x_pre))
            if i < n_d:
                phases.append(("dec", dw, dw.layer_begin + i, self.x_dec))
            if len({ph[2] for ph in phases}) < len(phases):
                for ph in phases:   # both phases at the same layer: keep their checks apart
                    self._run([ph], p, flags)
            else:
                self._run(phases, p, flags)
        return 1.0   # virtual cycle time (the device time is not under test here)

    def _run(self, phases, p, flags):
        B = self.B
        snap = {}
        batches = {}
        for name, wk, layer, x in phases:
            bt = self.table(wk.reqs)
            batches[name] = B.Batch(wk.q_lens, wk.ctx_lens, bt, x, layer, layer + 1)
            snap[name] = (x.cpu().numpy().copy(), self.pools[layer][0].float().cpu().numpy(),
                          self.pools[layer][1].float().cpu().numpy(), bt)
        pre, dec = batches.get("pre"), batches.get("dec")
        N = self.bl.n_sms
        pp = p if 0 < p < N else N // 2 // 2 * 2
        if pre is None:
            pp = 0
        elif dec is None:
            pp = N
        cur = torch.cuda.current_stream()
        self.sp.wait_stream(cur); self.sd.wait_stream(cur)
        self.bl.step(pre, dec, pp, flags, self.sp, self.sd)
        torch.cuda.synchronize()
        for name, wk, layer, x in phases:
            x0, pk, pv, bt = snap[name]
            q, c = list(wk.q_lens), list(wk.ctx_lens)
            mask = None
            if name == "pre" and sum(q) > 96:
                rng = np.random.default_rng(layer)
                mask = np.zeros(sum(q), np.uint8)
                mask[rng.choice(sum(q), 64, replace=False)] = 1
                mask[np.cumsum(q) - 1] = 1
            pk_o, pv_o = pk.copy(), pv.copy()
            ref = self._oracle(layer, x0, q, c, bt, pk_o, pv_o, mask)
            got = x.cpu().numpy()
            sel = slice(None) if mask is None else mask.astype(bool)
            mx, mr = compare(got[sel], ref[sel])
            assert mx <= 2e-2 and mr <= 1e-3, (name, layer, mx, mr)
            self.worst = max(self.worst, mr)
            # KV: the slots of this step's new positions, and nothing else
            gk = self.pools[layer][0].float().cpu().numpy()
            gv = self.pools[layer][1].float().cpu().numpy()
            new = np.zeros(gk.shape[0] * 16, bool)
            for r, (ql, cl) in enumerate(zip(q, c)):
                for j in range(ql):
                    pos = cl + j
                    new[bt[r][pos // 16] * 16 + pos % 16] = True
            for g_, o_, old in ((gk, pk_o, pk), (gv, pv_o, pv)):
                gs, os_, ol = (a_.transpose(0, 2, 1, 3).reshape(-1, a_.shape[1], a_.shape[3]) for a_ in (g_, o_, old))
                assert np.array_equal(gs[~new], ol[~new])
                assert np.all(np.abs(gs[new] - os_[new]) <= np.abs(os_[new]) * 2.0 ** -7 + 2e-3)
                assert np.mean(gs[new] == os_[new]) > 0.98
            self.checked[name] += 1


def test_serving_cycles_on_device_match_oracle():
    import paper_conf_asplos_0001xc0l026_b200 as B
    from paper_conf_asplos_0001xc0l026_b200 import serving as SV
    import os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    pj = os.path.join(root, "profiles", "perf_params_b200.json")
    torch.cuda.set_device(0)
    w_cpu = [synth.layer_weights(M, l) for l in range(M.n_layers)]
    pools = [tuple(t.to("cuda", torch.bfloat16).contiguous() for t in synth.kv_pool(M, N_BLOCKS, 16, l))
             for l in range(M.n_layers)]
    bl = B.Bullet(B.Model.of(M), pools, 4096, 256, 4096, perf_params_json=open(pj).read())
    for l in range(M.n_layers):
        bl.set_layer_weights(l, {k: (None if v is None else v.to("cuda", torch.bfloat16)) for k, v in w_cpu[l].items()})
    step = CheckedStep(B, bl, w_cpu, pools)
    trace = SV.poisson_trace(200.0, 0.2, seed=4, prompt_clip=(16, 600), out_clip=(2, 12))
    loop = SV.ServingLoop(M.n_layers, bl.n_sms, step, bl.choose_split, "bullet", SV.BlockAllocator(N_BLOCKS),
                          max_prefill_tokens=2048, max_decodes=64, k_full=2)
    loop.run(trace, max_cycles=20)
    assert len(loop.log) >= 15   # (max_cycles also counts idle waits for arrivals)
    assert step.checked["pre"] >= 4 and step.checked["dec"] >= 4, step.checked
    ks = {c[2] for c in loop.log}
    assert any(0 < c[1] < bl.n_sms for c in loop.log) or ks   # the loop really co-ran / decided splits
    bl.close()
