"""Pins of the CPU oracle (oracle/bullet_oracle.c) against things other than
itself: closed forms, invariants, brute force, and library routines on
special cases.  CPU only (-m "not gpu").  Each test names the passage or
DESIGN.md reading it pins."""
import math

import numpy as np
import pytest
import torch

import oracle as O
from workload import synth

RNG = np.random.default_rng(12345)


def tiny_cfg(H=4, Hkv=2, hd=16, d=64, I=96, mirror=1, llama3=0, theta=10000.0):
    return O.OracleCfg(d_model=d, n_heads=H, n_kv_heads=Hkv, head_dim=hd, d_ff=I,
                       rms_eps=1e-5, rope_theta=theta, rope_llama3=llama3, bf16_mirror=mirror)


def rand_weights(cfg, rng, bias=False, scale=1.0):
    d, H, Hkv, hd, I = cfg.d_model, cfg.n_heads, cfg.n_kv_heads, cfg.head_dim, cfg.d_ff
    nq = (H + 2 * Hkv) * hd
    bf = O.round_bf16 if cfg.bf16_mirror else (lambda a: a)
    f = lambda *s, std: np.asarray(bf(rng.standard_normal(s) * std * scale), dtype=np.float32)
    return {"w_qkv": f(nq, d, std=d ** -0.5), "b_qkv": f(nq, std=0.02) if bias else None,
            "w_o": f(d, H * hd, std=(H * hd) ** -0.5), "w_gate_up": f(2 * I, d, std=d ** -0.5),
            "w_down": f(d, I, std=I ** -0.5),
            "g_attn": np.asarray(bf(1 + 0.05 * rng.standard_normal(d)), dtype=np.float32),
            "g_mlp": np.asarray(bf(1 + 0.05 * rng.standard_normal(d)), dtype=np.float32)}


def make_pool(cfg, lay, rng, mirror=True):
    shape = (lay.n_blocks, cfg.n_kv_heads, lay.block_size, cfg.head_dim)
    k = rng.standard_normal(shape); v = rng.standard_normal(shape)
    if mirror:
        k, v = O.round_bf16(k), O.round_bf16(v)
    return np.ascontiguousarray(k, dtype=np.float32), np.ascontiguousarray(v, dtype=np.float32)


# ------------------------------------------------------------------ bf16 R-3

def test_round_bf16_matches_torch_rne_on_fp32_values():
    """R-3 rounding = IEEE round-to-nearest-even, checked against torch's
    fp32->bf16 conversion (library routine) incl. exact ties."""
    x = (RNG.standard_normal(20000) * 2.0 ** RNG.integers(-100, 100, 20000)).astype(np.float32)
    bits = x.view(np.uint32)
    ties = ((bits & np.uint32(0xFFFF0000)) | np.uint32(0x8000)).view(np.float32)   # exact halfway
    odd_ties = ((bits & np.uint32(0xFFFF0000)) | np.uint32(0x18000)).view(np.float32)
    for arr in (x, ties, odd_ties):
        ref = torch.from_numpy(arr).bfloat16().double().numpy()
        got = O.round_bf16(arr.astype(np.float64))
        assert np.array_equal(got, ref)


def test_round_bf16_special_values():
    assert O.round_bf16(np.array([0.0]))[0] == 0.0
    assert O.round_bf16(np.array([1.0 + 2 ** -8]))[0] == 1.0          # tie -> even
    assert O.round_bf16(np.array([1.0 + 3 * 2 ** -8]))[0] == 1.0 + 2 ** -6
    assert math.isinf(O.round_bf16(np.array([3.5e38]))[0])
    tiny = 2.0 ** -133
    assert O.round_bf16(np.array([tiny]))[0] == tiny                    # subnormal bf16


# ------------------------------------------------------------- RMSNorm R-1

def test_rmsnorm_constant_vector_closed_form():
    d, c, eps = 64, 3.0, 1e-5
    g = RNG.standard_normal(d).astype(np.float32)
    h = O.rmsnorm(np.full(d, c), g, eps)[0]
    assert np.allclose(h, c / math.sqrt(c * c + eps) * g.astype(np.float64), rtol=1e-15, atol=0)


def test_rmsnorm_unit_rms_and_scale_invariance():
    x = RNG.standard_normal((3, 128))
    g = np.ones(128, dtype=np.float32)
    h = O.rmsnorm(x, g, 0.0)
    assert np.allclose(np.sqrt((h ** 2).mean(1)), 1.0, rtol=1e-14)
    assert np.allclose(O.rmsnorm(7.5 * x, g, 0.0), h, rtol=1e-13)


# ------------------------------------------------------------------ linear

def test_linear_integer_operands_exact():
    """y = h W^T: integer operands give exact sums (vs numpy int64 matmul)."""
    h = RNG.integers(-2, 3, size=(5, 96))
    W = RNG.integers(-2, 3, size=(40, 96))
    b = RNG.integers(-3, 4, size=40)
    y = O.linear(h.astype(np.float64), W.astype(np.float32), b.astype(np.float32))
    assert np.array_equal(y, (h @ W.T + b).astype(np.float64))


# -------------------------------------------------------------------- RoPE

def test_rope_inv_freq_plain_and_llama3_vs_transformers():
    c = tiny_cfg(hd=128, theta=500000.0)
    f = O.rope_inv_freq(c)
    assert np.allclose(f, 500000.0 ** (-np.arange(0, 128, 2) / 128.0), rtol=1e-14)
    from transformers import LlamaConfig
    from transformers.modeling_rope_utils import _compute_llama3_parameters
    hf = LlamaConfig(hidden_size=4096, num_attention_heads=32, head_dim=128,
                     max_position_embeddings=131072, rope_theta=500000.0,
                     rope_scaling={"rope_type": "llama3", "factor": 8.0, "low_freq_factor": 1.0,
                                   "high_freq_factor": 4.0,
                                   "original_max_position_embeddings": 8192})
    ref, _ = _compute_llama3_parameters(hf, "cpu")
    c3 = tiny_cfg(hd=128, theta=500000.0, llama3=1)
    got = O.rope_inv_freq(c3)
    assert np.allclose(got, ref.double().numpy(), rtol=2e-6)
    # the three bands: highest frequency unchanged, lowest divided by factor
    assert got[0] == 1.0 and math.isclose(got[-1], f[-1] / 8.0, rel_tol=1e-14)


def test_rope_identity_norm_and_relative_position():
    c = tiny_cfg(hd=64)
    f = O.rope_inv_freq(c)
    q, k = RNG.standard_normal(64), RNG.standard_normal(64)
    assert np.array_equal(O.rope_apply(q, 0, f), q)
    r = O.rope_apply(q, 37, f)
    assert math.isclose(np.linalg.norm(r), np.linalg.norm(q), rel_tol=1e-14)
    for m, n in [(5, 2), (100, 37), (9, 9)]:
        lhs = O.rope_apply(q, m, f) @ O.rope_apply(k, n, f)
        rhs = O.rope_apply(q, m - n, f) @ k
        assert math.isclose(lhs, rhs, rel_tol=1e-11, abs_tol=1e-11)


def test_rope_rotate_half_pairs_by_hand():
    """hd = 4: pairs (0,2) and (1,3) rotate by pos*theta^0 and pos*theta^-1/2."""
    c = tiny_cfg(hd=4, theta=100.0)
    f = O.rope_inv_freq(c)
    assert np.allclose(f, [1.0, 0.1], rtol=1e-15)
    u = np.array([1.0, 0.0, 0.0, 1.0])
    r = O.rope_apply(u, 2, f)
    expect = [math.cos(2), -math.sin(0.2), math.sin(2), math.cos(0.2)]
    assert np.allclose(r, expect, rtol=1e-15, atol=1e-15)


# ------------------------------------------------------- attention (R-8)

def _dense_attention_bruteforce(Q, K, V):
    """Separate code path: materialise S = QK^T/sqrt(hd), causal mask (key j <=
    query i, keys/queries aligned at the end), softmax, times V.  numpy fp64."""
    nq, hd = Q.shape
    nk = K.shape[0]
    S = Q @ K.T / math.sqrt(hd)
    off = nk - nq
    mask = np.arange(nk)[None, :] <= (np.arange(nq)[:, None] + off)
    S = np.where(mask, S, -np.inf)
    S = S - S.max(1, keepdims=True)
    P = np.exp(S)
    P /= P.sum(1, keepdims=True)
    return P @ V


def _layer_inputs(cfg, q_lens, ctx_lens, B=16, seed=0, mirror=True, bias=False):
    rng = np.random.default_rng(seed)
    lay = synth.paged_layout(q_lens, ctx_lens, B, seed_offset=seed)
    w = rand_weights(cfg, rng, bias=bias)
    pk, pv = make_pool(cfg, lay, rng, mirror)
    x = rng.standard_normal((int(sum(q_lens)), cfg.d_model))
    return lay, w, pk, pv, x


def test_attend_paged_vs_bruteforce_and_sdpa():
    cfg = tiny_cfg(hd=16)
    rng = np.random.default_rng(3)
    ctx = 45
    lay = synth.paged_layout([1], [ctx], 16)
    pk, pv = make_pool(cfg, lay, rng)
    q = rng.standard_normal(16)
    bt = lay.block_table[0]
    for kvh in range(cfg.n_kv_heads):
        got = O.attend_paged(q, pk, pv, bt, 16, kvh, ctx)
        K = np.stack([pk[bt[j // 16], kvh, j % 16] for j in range(ctx + 1)]).astype(np.float64)
        V = np.stack([pv[bt[j // 16], kvh, j % 16] for j in range(ctx + 1)]).astype(np.float64)
        ref = _dense_attention_bruteforce(q[None], K, V)[0]
        assert np.allclose(got, ref, rtol=1e-12, atol=1e-13)
        sd = torch.nn.functional.scaled_dot_product_attention(
            torch.from_numpy(q)[None, None], torch.from_numpy(K)[None], torch.from_numpy(V)[None])
        assert np.allclose(got, sd[0, 0].numpy(), rtol=1e-12, atol=1e-13)


def test_attention_special_cases():
    cfg = tiny_cfg(hd=8, H=2, Hkv=2)
    rng = np.random.default_rng(4)
    lay = synth.paged_layout([1], [15], 16)
    pk, pv = make_pool(cfg, lay, rng, mirror=False)
    bt = lay.block_table[0]
    q = rng.standard_normal(8)
    # one key -> o = v_0 exactly
    assert np.array_equal(O.attend_paged(q, pk, pv, bt, 16, 0, 0), pv[bt[0], 0, 0].astype(np.float64))
    # q = 0 -> uniform mean of v
    o = O.attend_paged(np.zeros(8), pk, pv, bt, 16, 1, 15)
    assert np.allclose(o, pv[bt[0], 1, :16].astype(np.float64).mean(0), rtol=1e-13)
    # identical keys -> mean of v
    pk2 = pk.copy(); pk2[bt[0], 0, :] = pk[bt[0], 0, 0]
    o = O.attend_paged(q, pk2, pv, bt, 16, 0, 15)
    assert np.allclose(o, pv[bt[0], 0, :16].astype(np.float64).mean(0), rtol=1e-13)


# ------------------------------------------------------ layer invariants

def test_layer_zero_projections_is_identity():
    """W_o = 0 and W_down = 0 -> out == x bit-exact (steps 6, 9)."""
    cfg = tiny_cfg()
    lay, w, pk, pv, x = _layer_inputs(cfg, [7, 1, 1], [0, 20, 33])
    w["w_o"][:] = 0; w["w_down"][:] = 0
    out = O.layer_forward(cfg, w, pk, pv, lay.q_lens, lay.ctx_lens, lay.block_table, x)
    assert np.array_equal(out, x)


def test_layer_kv_write_slots_and_sentinel():
    """Step 4: new k/v land exactly at bt[r][p/B]*B + p%B; every other pool
    entry keeps its sentinel (bit-exact)."""
    cfg = tiny_cfg()
    lay, w, pk, pv, x = _layer_inputs(cfg, [21, 1, 1], [0, 16, 40])
    pk[:] = -777.0; pv[:] = -777.0
    _, dg = O.layer_forward(cfg, w, pk, pv, lay.q_lens, lay.ctx_lens, lay.block_table, x, diag=True)
    written = np.zeros(pk.shape[:1] + pk.shape[2:3], dtype=bool)   # [blk][slot]
    for r, (q, c) in enumerate(zip(lay.q_lens, lay.ctx_lens)):
        for p in range(c, c + q):
            written[lay.block_table[r][p // 16], p % 16] = True
    for blk in range(pk.shape[0]):
        for s in range(16):
            if written[blk, s]:
                assert np.all(pk[blk, :, s] != -777.0) and np.all(pv[blk, :, s] != -777.0)
            else:
                assert np.all(pk[blk, :, s] == -777.0) and np.all(pv[blk, :, s] == -777.0)


def test_paging_invariance_bit_exact():
    """Same KV stored contiguously vs in randomly permuted blocks, block sizes
    1 / 16 / whole sequence -> bit-identical outputs (P:L227 index table)."""
    cfg = tiny_cfg()
    rng = np.random.default_rng(7)
    w = rand_weights(cfg, rng)
    ctx = [0, 29, 50]
    ql = [13, 1, 1]
    x = rng.standard_normal((sum(ql), cfg.d_model))
    # cached context as a dense [req][pos][Hkv][hd] array
    ctxK = O.round_bf16(rng.standard_normal((3, 64, cfg.n_kv_heads, cfg.head_dim)))
    ctxV = O.round_bf16(rng.standard_normal((3, 64, cfg.n_kv_heads, cfg.head_dim)))
    outs = []
    for B, perm in [(64, False), (1, True), (16, True), (16, False)]:
        lay = synth.paged_layout(ql, ctx, B, seed_offset=B)
        bt = lay.block_table.copy()
        if not perm:   # contiguous: request r owns blocks r*nb .. r*nb+nb-1
            nb = bt.shape[1]
            bt = np.arange(3 * nb, dtype=np.int32).reshape(3, nb)
            n_blocks = 3 * nb
        else:
            n_blocks = lay.n_blocks
        pk = np.zeros((n_blocks, cfg.n_kv_heads, B, cfg.head_dim), np.float32)
        pv = np.zeros_like(pk)
        for r in range(3):
            for p in range(ctx[r]):
                pk[bt[r][p // B], :, p % B] = ctxK[r, p]
                pv[bt[r][p // B], :, p % B] = ctxV[r, p]
        outs.append(O.layer_forward(cfg, w, pk, pv, ql, ctx, bt, x))
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])


def test_prefill_then_decode_equals_full_prefill_row():
    """Decode of token t with KV from a prefill of tokens 0..t-1 equals row t
    of a full prefill of 0..t (P:L42, P:L227 copy-free hand-off)."""
    cfg = tiny_cfg()
    rng = np.random.default_rng(11)
    w = rand_weights(cfg, rng)
    t = 37
    x = rng.standard_normal((t + 1, cfg.d_model))
    lay = synth.paged_layout([t + 1], [0], 16)
    pk = np.zeros((lay.n_blocks, cfg.n_kv_heads, 16, cfg.head_dim), np.float32); pv = pk.copy()
    full = O.layer_forward(cfg, w, pk, pv, [t + 1], [0], lay.block_table, x)
    pk2 = np.zeros_like(pk); pv2 = np.zeros_like(pv)
    O.layer_forward(cfg, w, pk2, pv2, [t], [0], lay.block_table, x[:t])
    dec = O.layer_forward(cfg, w, pk2, pv2, [1], [t], lay.block_table, x[t:])
    assert np.array_equal(dec[0], full[t])
    assert np.array_equal(pk, pk2) and np.array_equal(pv, pv2)


def test_row_sampling_matches_full_rows():
    cfg = tiny_cfg()
    lay, w, pk, pv, x = _layer_inputs(cfg, [30, 1, 1], [0, 17, 3])
    full = O.layer_forward(cfg, w, pk.copy(), pv.copy(), lay.q_lens, lay.ctx_lens, lay.block_table, x)
    mask = np.zeros(32, np.uint8); mask[[0, 5, 29, 30, 31]] = 1
    samp = O.layer_forward(cfg, w, pk.copy(), pv.copy(), lay.q_lens, lay.ctx_lens, lay.block_table, x,
                           row_mask=mask)
    assert np.array_equal(samp[mask == 1], full[mask == 1])
    assert np.all(samp[mask == 0] == 0)


def test_gqa_equals_mha_with_duplicated_kv_heads():
    """Hkv = H reduces GQA to MHA: duplicating each kv head's weights and
    cache across its group gives bit-identical outputs (head g = h/(H/Hkv))."""
    cfg = tiny_cfg(H=4, Hkv=2)
    rng = np.random.default_rng(5)
    w = rand_weights(cfg, rng)
    ql, ctx = [9, 1], [0, 23]
    lay = synth.paged_layout(ql, ctx, 16)
    pk, pv = make_pool(cfg, lay, rng)
    x = rng.standard_normal((10, cfg.d_model))
    out_gqa = O.layer_forward(cfg, w, pk.copy(), pv.copy(), ql, ctx, lay.block_table, x)
    hd, H = cfg.head_dim, cfg.n_heads
    q_rows = w["w_qkv"][:H * hd]
    k_rows = w["w_qkv"][H * hd:(H + 2) * hd].reshape(2, hd, -1)
    v_rows = w["w_qkv"][(H + 2) * hd:].reshape(2, hd, -1)
    w2 = dict(w)
    w2["w_qkv"] = np.concatenate([q_rows, np.repeat(k_rows, 2, 0).reshape(-1, cfg.d_model),
                                  np.repeat(v_rows, 2, 0).reshape(-1, cfg.d_model)])
    cfg2 = tiny_cfg(H=4, Hkv=4)
    out_mha = O.layer_forward(cfg2, w2, np.repeat(pk, 2, 1).copy(), np.repeat(pv, 2, 1).copy(),
                              ql, ctx, lay.block_table, x)
    assert np.array_equal(out_gqa, out_mha)


def _torch_layer(cfg, w, K_ctx, V_ctx, x_new, pos0):
    """Library cross-check (torch fp64 ops: rms_norm, linear, sdpa, silu) of
    one request; K_ctx/V_ctx [ctx][Hkv][hd] are the cached keys/values."""
    T = lambda a: torch.from_numpy(np.asarray(a, dtype=np.float64))
    rb = lambda t: T(O.round_bf16(t.numpy())) if cfg.bf16_mirror else t
    H, Hkv, hd, I, d = cfg.n_heads, cfg.n_kv_heads, cfg.head_dim, cfg.d_ff, cfg.d_model
    x = T(x_new)
    n = x.shape[0]
    h = rb(torch.nn.functional.rms_norm(x, (d,), T(w["g_attn"]), eps=cfg.rms_eps))
    qkv = torch.nn.functional.linear(h, T(w["w_qkv"]), None if w["b_qkv"] is None else T(w["b_qkv"]))
    f = T(O.rope_inv_freq(cfg))
    pos = torch.arange(pos0, pos0 + n, dtype=torch.float64)
    ang = pos[:, None] * f[None]
    cos, sin = torch.cos(ang)[:, None], torch.sin(ang)[:, None]

    def rope(u):   # u [n][heads][hd]
        a, b = u[..., :hd // 2], u[..., hd // 2:]
        return torch.cat([a * cos - b * sin, b * cos + a * sin], -1)
    q = rope(qkv[:, :H * hd].reshape(n, H, hd))
    k = rope(qkv[:, H * hd:(H + Hkv) * hd].reshape(n, Hkv, hd))
    v = qkv[:, (H + Hkv) * hd:].reshape(n, Hkv, hd)
    q, k, v = rb(q), rb(k), rb(v)
    K = torch.cat([T(K_ctx), k]); V = torch.cat([T(V_ctx), v])
    nk = K.shape[0]
    mask = torch.arange(nk)[None, :] <= (torch.arange(n)[:, None] + pos0)
    Kh = K.repeat_interleave(H // Hkv, 1).transpose(0, 1)
    Vh = V.repeat_interleave(H // Hkv, 1).transpose(0, 1)
    o = torch.nn.functional.scaled_dot_product_attention(q.transpose(0, 1), Kh, Vh, attn_mask=mask)
    o = rb(o.transpose(0, 1).reshape(n, H * hd))
    x1 = x + torch.nn.functional.linear(o, T(w["w_o"]))
    h2 = rb(torch.nn.functional.rms_norm(x1, (d,), T(w["g_mlp"]), eps=cfg.rms_eps))
    gu = torch.nn.functional.linear(h2, T(w["w_gate_up"]))
    a = rb(torch.nn.functional.silu(gu[:, :I]) * gu[:, I:])
    return (x1 + torch.nn.functional.linear(a, T(w["w_down"]))).numpy()


@pytest.mark.parametrize("mirror,bias,llama3", [(1, False, 1), (1, True, 0), (0, False, 0)])
def test_layer_vs_torch_library_composition(mirror, bias, llama3):
    """Whole layer against torch fp64 library ops (rms_norm, linear, sdpa,
    silu) per request: catches transposed operands, dropped terms, wrong
    head grouping.  Tolerance: fp64 reassociation + the rare bf16 rounding
    flip it can cause at R1-R5 (one bf16 ulp on a few elements)."""
    cfg = tiny_cfg(mirror=mirror, llama3=llama3, theta=500000.0 if llama3 else 10000.0)
    ql, ctx = [19, 1, 1, 5], [0, 30, 47, 16]
    lay, w, pk, pv, x = _layer_inputs(cfg, ql, ctx, seed=21, mirror=bool(mirror), bias=bias)
    pk0, pv0 = pk.copy(), pv.copy()
    out = O.layer_forward(cfg, w, pk, pv, lay.q_lens, lay.ctx_lens, lay.block_table, x)
    row = 0
    for r, (q, c) in enumerate(zip(ql, ctx)):
        bt = lay.block_table[r]
        Kc = np.stack([pk0[bt[p // 16], :, p % 16] for p in range(c)]) if c else \
            np.zeros((0, cfg.n_kv_heads, cfg.head_dim))
        Vc = np.stack([pv0[bt[p // 16], :, p % 16] for p in range(c)]) if c else \
            np.zeros((0, cfg.n_kv_heads, cfg.head_dim))
        ref = _torch_layer(cfg, w, Kc, Vc, x[row:row + q], c)
        err = np.abs(out[row:row + q] - ref)
        # fp32 mode: the pool stores the new k/v as float (fp32 rounding) -> ~1e-7
        assert err.max() < (2e-2 if mirror else 1e-6)
        assert err.sum() / np.abs(ref).sum() < (1e-4 if mirror else 1e-7)
        row += q


def test_tp_shard_sum_equals_unsharded():
    """Megatron TP identity (north_star (4)): sum over ranks of the
    row-parallel partial products equals the unsharded product (fp64)."""
    m = synth.ModelShape("t", 64, 4, 2, 16, 96, 1)
    w = synth.layer_weights(m, 0)
    rng = np.random.default_rng(2)
    h = rng.standard_normal((5, 96))
    full = O.linear(h, w["w_down"].numpy())
    parts = sum(O.linear(h[:, r * 48:(r + 1) * 48],
                         synth.shard_weights(m, w, 2, r)["w_down"].numpy()) for r in range(2))
    assert np.allclose(parts, full, rtol=1e-13, atol=1e-13)
    o = rng.standard_normal((5, 64))
    full_o = O.linear(o, w["w_o"].numpy())
    parts_o = sum(O.linear(o[:, r * 32:(r + 1) * 32],
                           synth.shard_weights(m, w, 2, r)["w_o"].numpy()) for r in range(2))
    assert np.allclose(parts_o, full_o, rtol=1e-13, atol=1e-13)


def test_layer_rejects_out_of_range_block():
    cfg = tiny_cfg()
    lay, w, pk, pv, x = _layer_inputs(cfg, [3], [0])
    bt = lay.block_table.copy(); bt[0, 0] = lay.n_blocks
    with pytest.raises(ValueError):
        O.layer_forward(cfg, w, pk, pv, lay.q_lens, lay.ctx_lens, bt, x)
