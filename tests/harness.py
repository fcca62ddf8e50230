"""Test harness: builds the same seeded layer-step inputs for the CUDA path
(through the C ABI binding) and for the CPU oracle.  Test-only code."""
from __future__ import annotations

import numpy as np
import torch

import oracle as O
from workload import synth


def oracle_cfg(m: synth.ModelShape) -> O.OracleCfg:
    return O.OracleCfg(d_model=m.d_model, n_heads=m.n_heads, n_kv_heads=m.n_kv_heads,
                       head_dim=m.head_dim, d_ff=m.d_ff, rms_eps=m.rms_eps, rope_theta=m.rope_theta,
                       rope_llama3=m.rope_llama3, rope_factor=m.rope_factor,
                       rope_low_freq=m.rope_low_freq, rope_high_freq=m.rope_high_freq,
                       rope_orig_max_pos=m.rope_orig_max_pos,
                       bf16_mirror=1 if m.dtype == "bf16" else 0)


def phase_streams():
    """Two fresh streams for bullet_step, ordered after everything already
    enqueued on the current stream (the inputs' host->device copies): the
    library orders nothing the caller enqueued elsewhere (include/bullet.h)."""
    cur = torch.cuda.current_stream()
    sp, sd = torch.cuda.Stream(), torch.cuda.Stream()
    sp.wait_stream(cur)
    sd.wait_stream(cur)
    return sp, sd


class Setup:
    """Model weights + KV pools + one co-run step's batches, on CPU (oracle)
    and on the GPU (product)."""

    def __init__(self, m: synth.ModelShape, prefill_lens, decode_ctx, n_layers=1,
                 max_position=None, perf_params_json=None, slack=0.25):
        import paper_conf_asplos_0001xc0l026_b200 as B
        self.B = B
        self.m = m
        self.n_layers = n_layers
        self.prefill_lens = list(prefill_lens)
        self.decode_ctx = list(decode_ctx)
        q = self.prefill_lens + [1] * len(self.decode_ctx)
        c = [0] * len(self.prefill_lens) + self.decode_ctx
        self.lay = synth.paged_layout(q, c, 16, slack=slack)
        self.n_pre = len(self.prefill_lens)
        self.w_cpu = [synth.layer_weights(m, l) for l in range(n_layers)]
        self.pool_cpu = [synth.kv_pool(m, self.lay.n_blocks, 16, l) for l in range(n_layers)]
        td = torch.bfloat16 if m.dtype == "bf16" else torch.float32
        self.w_gpu = [{k: (None if v is None else v.to("cuda", td)) for k, v in w.items()}
                      for w in self.w_cpu]
        self.pool_gpu = [(k.to("cuda", td).contiguous(), v.to("cuda", td).contiguous())
                         for k, v in self.pool_cpu]
        n_p, n_d = sum(self.prefill_lens), len(self.decode_ctx)
        self.x_pre = synth.hidden(max(n_p, 0), m.d_model, seed_offset=0)
        self.x_dec = synth.hidden(max(n_d, 0), m.d_model, seed_offset=1)
        maxpos = max_position or (max(q[i] + c[i] for i in range(len(q))) + 16)
        self.bl = B.Bullet(B.Model.of(m), self.pool_gpu, max_prefill_tokens=max(n_p, 1),
                           max_decode_tokens=max(n_d, 1), max_position=maxpos,
                           perf_params_json=perf_params_json)
        for l in range(n_layers):
            self.bl.set_layer_weights(l, self.w_gpu[l])

    def batches(self, layer_begin=0, layer_end=None):
        B = self.B
        le = self.n_layers if layer_end is None else layer_end
        bt = self.lay.block_table
        pre = dec = None
        if self.n_pre:
            pre = B.Batch(self.prefill_lens, [0] * self.n_pre, bt[:self.n_pre],
                          self.x_pre.cuda().contiguous(), layer_begin, le)
        if self.decode_ctx:
            dec = B.Batch([1] * len(self.decode_ctx), self.decode_ctx, bt[self.n_pre:],
                          self.x_dec.cuda().contiguous(), layer_begin, le)
        return pre, dec

    def oracle(self, row_mask_pre=None, layers=None):
        """Oracle outputs (fp64) of both phases through `layers` layers,
        fp32-rounded residual stream between layers (storage mirror)."""
        cfg = oracle_cfg(self.m)
        layers = self.n_layers if layers is None else layers
        out = {}
        for name, x, q, c, bt, mask in (
                ("pre", self.x_pre, self.prefill_lens, [0] * self.n_pre,
                 self.lay.block_table[:self.n_pre], row_mask_pre),
                ("dec", self.x_dec, [1] * len(self.decode_ctx), self.decode_ctx,
                 self.lay.block_table[self.n_pre:], None)):
            if not q:
                continue
            xs = x.double().numpy()
            for l in range(layers):
                pk = self.pool_cpu[l][0].numpy().copy(); pv = self.pool_cpu[l][1].numpy().copy()
                w = {k: (None if v is None else v.numpy()) for k, v in self.w_cpu[l].items()}
                o = O.layer_forward(cfg, w, pk, pv, q, c, bt, xs, row_mask=mask if l == layers - 1 else None)
                xs = o.astype(np.float32).astype(np.float64) if l < layers - 1 else o
            out[name] = xs
        return out


def oracle_layer(S, layer, x_pre, x_dec, row_mask_pre=None):
    """One oracle layer step from given fp32 inputs (e.g. the GPU's output of
    the previous layer): per-step parity (DESIGN R-4c)."""
    cfg = oracle_cfg(S.m)
    w = {k: (None if v is None else v.numpy()) for k, v in S.w_cpu[layer].items()}
    out = {}
    for name, x, q, c, bt, mask in (
            ("pre", x_pre, S.prefill_lens, [0] * S.n_pre, S.lay.block_table[:S.n_pre], row_mask_pre),
            ("dec", x_dec, [1] * len(S.decode_ctx), S.decode_ctx, S.lay.block_table[S.n_pre:], None)):
        if not q:
            continue
        pk = S.pool_cpu[layer][0].numpy().copy(); pv = S.pool_cpu[layer][1].numpy().copy()
        out[name] = O.layer_forward(cfg, w, pk, pv, q, c, bt, np.asarray(x, dtype=np.float64),
                                    row_mask=mask)
    return out


def compare(got: np.ndarray, ref: np.ndarray):
    """(max-abs error, normalized-L1 mean-rel error) — DESIGN.md R-4."""
    err = np.abs(got.astype(np.float64) - ref)
    return float(err.max()), float(err.sum() / max(np.abs(ref).sum(), 1e-300))
