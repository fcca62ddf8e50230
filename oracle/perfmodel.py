"""TEST INFRASTRUCTURE ONLY — plain reading of Bullet's performance estimator
and SLO-aware split decision (§3.2-§3.3), for checking the product's
``bullet_model_predict`` / ``bullet_choose_split`` (C++ in libbullet.so).

Written straight from the paper, in its order and notation:
  Eq. 1  s = 1 - g / (M * ceil(g / M))                          P:L57-59 (§2.2.1)
  Eq. 2  t_i = max(c_i/C * M/(m_i d_c p_c), b_i/B * M/(m_i d_b p_b)) * (1-s_i)^-1
                                                                 P:L137-141 (§3.2.1)
  T_m = sum_i t_i over the kernels of one layer                  P:L149 (§3.2.2)
  Alg. 1 case split, decode-SM search, decode pause
Readings of garbled / silent points (R-11 .. R-18) are marked
"Reading R-nn" where they are used.  The per-kernel (c_i, b_i, g_i) inventory
describes OUR kernels; its tile sizes come from the params
dict, the same JSON the product loads.
"""
from __future__ import annotations

import math

# ------------------------------------------------------------------ Eq. 1

def wave_idle(g: int, M: int) -> float:
    """Eq. 1: idle SM-cycle ratio of g thread blocks on M SMs."""
    if g <= 0 or M <= 0:
        return 0.0
    w = math.ceil(g / M)
    return 1.0 - g / (M * w)


# ------------------------------------------------------------------ Eq. 2

def interp(table: dict, m: float) -> float:
    """Piecewise-linear d(m) through the fitted points (Reading R-12: the
    decay factors are functions of the SM count, P:L139 'non-linear')."""
    ms, vs = table["m"], table["v"]
    if m <= ms[0]:
        return vs[0]
    for i in range(1, len(ms)):
        if m <= ms[i]:
            f = (m - ms[i - 1]) / (ms[i] - ms[i - 1])
            return vs[i - 1] + f * (vs[i] - vs[i - 1])
    return vs[-1]


def kernel_time(c, b, C, B, M, m, d_c, d_b, p_c, p_b, s) -> float:
    """Eq. 2: seconds for c flops and b bytes on m of M SMs."""
    tc = c / C * M / (m * d_c * p_c)
    tb = b / B * M / (m * d_b * p_b)
    return max(tc, tb) / (1.0 - s)


# ------------------------------------------------ per-kernel (c_i, b_i, g_i)

def layer_kernels(shape: dict, P: dict, m: int) -> list:
    """(name, c_i flops, b_i bytes, g_i work units, occupancy) of one layer
    of one phase on m SMs.  ``shape``: d, H, Hkv, hd, I, elt (bytes per
    stored element: 2 bf16 / 4 fp32), q_lens (new tokens per request),
    ctx_lens (cached tokens per request).  DESIGN.md §5 lists the same."""
    d, H, Hkv, hd, I, e = (shape[k] for k in ("d", "H", "Hkv", "hd", "I", "elt"))
    q_lens, ctx_lens = shape["q_lens"], shape["ctx_lens"]
    n = sum(q_lens)
    if n == 0:
        return []
    nq = (H + 2 * Hkv) * hd
    T = P["tiles"]
    bm, bn, bk = T["gemm_bm"], T["gemm_bn"], T["gemm_bk"]
    rows = T["rows_per_unit"]
    occ_g, occ_a, occ_e = P["occ"]["gemm"], P["occ"]["attn"], P["occ"]["elem"]

    def gemm(name, K, N, extra_bytes):
        tiles = math.ceil(n / bm) * math.ceil(N / bn)
        splits = max(1, min(math.ceil(m * occ_g / tiles), K // (bk * T["min_k_blocks"])))
        return (name, 2.0 * n * K * N, e * (K * N + n * K) + extra_bytes, tiles * splits, occ_g)

    pairs = sum(q * c + q * (q + 1) // 2 for q, c in zip(q_lens, ctx_lens))   # keys <= position
    keys = sum(c + q for q, c in zip(q_lens, ctx_lens))
    if max(q_lens) > 1:     # prefill-style: q tiles x heads
        attn_units = sum(math.ceil(q / T["attn_bq"]) for q in q_lens) * H
    else:                   # decode: one unit per (request, kv head)
        attn_units = len(q_lens) * Hkv
    if e == 2 and hd == 128:   # bf16: RoPE + KV append fused into the QKV GEMM epilogue
        name, c, b, g, occ = gemm("qkv", d, nq, e * n * nq)
        qkv = [(name, c + 6.0 * n * (H + Hkv) * hd, b, g, occ)]
    else:
        qkv = [gemm("qkv", d, nq, 4 * n * nq),
               ("rope_kv", 6.0 * n * (H + Hkv) * hd, 4 * n * nq + e * n * nq, math.ceil(n / rows), occ_e)]
    ks = [
        ("rmsnorm1", 4.0 * n * d, 4 * n * d + e * n * d + e * d, math.ceil(n / rows), occ_e),
        *qkv,
        ("attn", 4.0 * hd * H * pairs, 2 * e * Hkv * hd * keys + 2 * e * n * H * hd, attn_units, occ_a),
        gemm("o_proj", H * hd, d, 8 * n * d),
        ("rmsnorm2", 4.0 * n * d, 4 * n * d + e * n * d + e * d, math.ceil(n / rows), occ_e),
        gemm("gate_up", d, 2 * I, e * n * I),
        gemm("down", I, d, 8 * n * d),
    ]
    return ks


def layer_time(shape: dict, P: dict, m: int, corun_m: int) -> float:
    """T_m = sum_i t_i in seconds for one layer of one phase on m
    SMs; the contention factors p_c, p_b apply only when a co-runner holds
    corun_m > 0 SMs (Reading R-11: one bandwidth factor p_b)."""
    if m <= 0:
        return math.inf
    M = P["M"]
    C, B = P["C_tflops"] * 1e12, P["B_gbs"] * 1e9
    d_c, d_b = interp(P["d_c"], m), interp(P["d_b"], m)
    # R-12b: the attention kernel's own decay tables (default: the same)
    d_ca = interp(P["d_c_attn"], m) if "d_c_attn" in P else d_c
    d_ba = interp(P["d_b_attn"], m) if "d_b_attn" in P else d_b
    # R-11/R-12: co-location factors, a constant or piecewise linear in the
    # kernel's own SM count m (fitted from co-run points, like d_c, d_b)
    def co(v):
        return interp(v, m) if isinstance(v, dict) else v
    p_c, p_b = (co(P["p_c"]), co(P["p_b"])) if corun_m > 0 else (1.0, 1.0)
    total = 0.0
    for name, c, b, g, occ in layer_kernels(shape, P, m):
        s = wave_idle(g, m * occ)          # Reading R-13: M := m_i x CTAs per SM
        dc, db = (d_ca, d_ba) if name == "attn" else (d_c, d_b)
        total += kernel_time(c, b, C, B, M, m, dc, db, p_c, p_b, s)
    # online level calibration per phase class (P:L195 feedback; default 1)
    return total * (P.get("scale_pre", 1.0) if max(shape["q_lens"], default=0) > 1 else P.get("scale_dec", 1.0))


# ------------------------------------------------------------ Alg. 1 reading

def p90(values, pct=0.9):
    """Nearest-rank percentile (Reading R-14): sorted[ceil(pct*n) - 1]."""
    if not values:
        return 0.0
    v = sorted(values)
    return v[max(0, math.ceil(pct * len(v)) - 1)]


def _phase_shape(model: dict, q_lens, ctx_lens):
    s = dict(model)
    s["q_lens"], s["ctx_lens"] = list(q_lens), list(ctx_lens)
    return s


def evaluate_split(P, model, state, slo, u, v):
    """Predicted P90 TTFT and TPOT ratios (value / SLO) for split (u, v).
    u = prefill SMs, v = decode SMs; u = N, v = 0 is the decode pause."""
    N, L, lk = P["M"], state["total_layers"], state["layers_done"]
    pre = _phase_shape(model, state["prefill_lens"], [0] * len(state["prefill_lens"]))
    dec = _phase_shape(model, [1] * len(state["decode_tokens"]),
                       [int(math.floor(state["decode_mean_ctx"] + 0.5))] * len(state["decode_tokens"]))
    ms = 1e3
    t_p = layer_time(pre, P, u, v) * ms if state["prefill_lens"] else 0.0
    rem = t_p * (L - lk)                                   # Alg. 1 line 3
    ttft = []
    for ln, q in zip(state["prefill_lens"], state["prefill_waited_ms"]):
        ttft.append((rem + q) / (slo["ttft_norm_ms_per_tok"] * ln))         # line 4-5 (R-18)
    for ln, q in zip(state["pending_lens"], state["pending_waited_ms"]):
        own = layer_time(_phase_shape(model, [ln], [0]), P, u, v) * ms * L   # R-15 (our addition)
        ttft.append((q + rem + own) / (slo["ttft_norm_ms_per_tok"] * ln))   # line 6-7
    tpot = []
    if state["decode_tokens"]:
        if v > 0:
            t_iter = layer_time(dec, P, v, u) * ms * L
        else:   # pause: wait one prefill layer cycle, then an iteration on v_k SMs alone
            t_iter = layer_time(pre, P, N, 0) * ms + layer_time(dec, P, state["v_k"], 0) * ms * L
        for o, dlat in zip(state["decode_tokens"], state["decode_elapsed_ms"]):
            tpot.append(((dlat + t_iter) / (o + 1)) / slo["tpot_ms"])      # lines 8-10 (R-14)
    pct = slo.get("percentile", 0.9)
    return p90(ttft, pct), p90(tpot, pct), t_p


GAIN_TOL = 0.06   # R-23: the model's resolution for the gain objective (held-out MRE ~6 %)


def candidates(P, slo, gran):
    """Decode SM counts v (prefill gets N - v) with v >= v_min and u >= gran."""
    N = P["M"]
    return [v for v in range(slo["v_min"], N - gran + 1) if v % gran == 0 or v == slo["v_min"]]


def choose_split(P, model, state, slo, gran=2):
    """Alg. 1 + the §3.3.3 search, Reading R-14..R-17.
    Returns (prefill_sm_count, decode_layer_steps)."""
    N, L = P["M"], state["total_layers"]
    has_pre = bool(state["prefill_lens"]) or bool(state["pending_lens"])
    if not state["decode_tokens"]:
        return N, 0
    if not has_pre:
        return 0, L
    cands = candidates(P, slo, gran)
    ev = {v: evaluate_split(P, model, state, slo, N - v, v) for v in cands}
    vk = min(cands, key=lambda v: (abs(v - state["v_k"]), v))   # current split, snapped
    ttft_k, tpot_k, _ = ev[vk]
    ok_t, ok_d = ttft_k <= 1.0, tpot_k <= 1.0

    def reduce_decode():
        feas = [v for v in cands if v <= vk and ev[v][0] <= 1.0 and ev[v][1] <= 1.0]
        if feas:
            return min(feas)
        pt, pd, _ = evaluate_split(P, model, state, slo, N, 0)
        if pd <= 1.0:
            return 0                                   # pause decode
        return min(cands)                              # v_min

    def reduce_prefill():
        feas = [v for v in cands if v >= vk and ev[v][1] <= 1.0]
        if feas:
            return min(feas)
        return min(cands, key=lambda v: (ev[v][1], v))

    def balanced():
        return min(cands, key=lambda v: (max(ev[v][0], ev[v][1]), v))   # R-16, tie -> larger u

    def max_throughput_t():
        # R-21 (objective 1, "meet stringent SLO requirements while
        # maximizing throughput"): among the SLO-feasible splits, the most
        # predicted tokens per ms; ties to the larger prefill share
        dec = _phase_shape(model, [1] * len(state["decode_tokens"]),
                           [int(math.floor(state["decode_mean_ctx"] + 0.5))] * len(state["decode_tokens"]))
        n_pre = float(sum(state["prefill_lens"]))
        best, best_t = None, -1.0
        for v in cands:
            if ev[v][0] > 1.0 or ev[v][1] > 1.0:
                continue
            t_p, t_d = ev[v][2], layer_time(dec, P, v, N - v) * 1e3
            k = max(1, int(math.floor(t_p / t_d + 0.5))) if t_d > 0 else 1
            cyc = max(t_p, k * t_d)
            tput = (n_pre + len(state["decode_tokens"]) * k) / cyc if cyc > 0 else 0.0
            if tput > best_t:
                best, best_t = v, tput
        return best, best_t

    def timesliced():
        # R-22: one prefill layer then k_ts decode layer-steps, both alone on
        # all N SMs, k_ts = round(t_p / t_d); Alg. 1 l.3-10 on the cycle time;
        # returns (k_ts, tokens per ms), k_ts = 0 when an SLO is missed
        pre = _phase_shape(model, list(state["prefill_lens"]), [0] * len(state["prefill_lens"]))
        dec = _phase_shape(model, [1] * len(state["decode_tokens"]),
                           [int(math.floor(state["decode_mean_ctx"] + 0.5))] * len(state["decode_tokens"]))
        tp = layer_time(pre, P, N, 0) * 1e3 if state["prefill_lens"] else 0.0
        td = layer_time(dec, P, N, 0) * 1e3
        if tp <= 0.0 or td <= 0.0:
            return 0, -1.0
        k = max(1, int(math.floor(tp / td + 0.5)))
        cyc = tp + k * td
        rem = cyc * (L - state["layers_done"])
        ttft = [(rem + q) / (slo["ttft_norm_ms_per_tok"] * ln)
                for ln, q in zip(state["prefill_lens"], state["prefill_waited_ms"])]
        for ln, q in zip(state["pending_lens"], state["pending_waited_ms"]):
            own = layer_time(_phase_shape(model, [ln], [0]), P, N, 0) * 1e3 * L
            ttft.append((q + rem + own) / (slo["ttft_norm_ms_per_tok"] * ln))
        it = cyc * L / k
        tpot = [((dlat + it) / (o + 1)) / slo["tpot_ms"]
                for o, dlat in zip(state["decode_tokens"], state["decode_elapsed_ms"])]
        pct = slo.get("percentile", 0.9)
        if p90(ttft, pct) > 1.0 or p90(tpot, pct) > 1.0:
            return 0, -1.0
        return k, (float(sum(state["prefill_lens"])) + len(state["decode_tokens"]) * k) / cyc

    def max_gain():
        # R-23 (objective 2): among SLO-feasible splits and k in {floor(r),
        # floor(r) + 1}, r = t_p / t_d (k >= 1), the largest predicted gain
        # (t_p(N) + k t_d(N)) / max(t_p(u), k t_d(v)) of co-running the cycle
        # over time-slicing the same work; ties: larger gain, then larger
        # prefill share (smaller v), then smaller k
        pre = _phase_shape(model, list(state["prefill_lens"]), [0] * len(state["prefill_lens"]))
        dec = _phase_shape(model, [1] * len(state["decode_tokens"]),
                           [int(math.floor(state["decode_mean_ctx"] + 0.5))] * len(state["decode_tokens"]))
        tpN = layer_time(pre, P, N, 0) * 1e3 if state["prefill_lens"] else 0.0
        tdN = layer_time(dec, P, N, 0) * 1e3
        cs = []
        for v in cands:
            if ev[v][0] > 1.0 or ev[v][1] > 1.0:
                continue
            t_p, t_d = ev[v][2], layer_time(dec, P, v, N - v) * 1e3
            if t_d <= 0:
                continue
            k0 = max(1, int(math.floor(t_p / t_d)))
            for k in (k0, k0 + 1):
                cs.append((v, k, (tpN + k * tdN) / max(t_p, k * t_d)))
        if not cs:
            return (None, 1), -1.0
        best_g = max(c[2] for c in cs)
        # gains within GAIN_TOL of the best are within the model's resolution:
        # the larger prefill share wins, then the larger gain, then smaller k
        near = [c for c in cs if c[2] >= (1.0 - GAIN_TOL) * best_g]
        v, k, _ = min(near, key=lambda c: (c[0], -c[2], c[1]))
        return (v, k), best_g

    if ok_t and ok_d and slo.get("objective", 0) == 2:
        (vb, kb), g = max_gain()
        if vb is not None and g > 1.0:
            return N - vb, kb
        k_ts, _ = timesliced()
        if k_ts > 0:
            return N, k_ts                             # co-running does not pay: time-sliced cycle
        if vb is not None:
            return N - vb, kb
        v = reduce_decode()
    elif ok_t and ok_d and slo.get("objective", 0) == 1:
        vb, t_co = max_throughput_t()                  # R-21
        k_ts, t_ts = timesliced()                      # R-22
        if k_ts > 0 and t_ts > t_co:
            return N, k_ts                             # time-sliced cycle (p = N, k > 0)
        v = vb if vb is not None else reduce_decode()
    elif ok_t and ok_d:
        v = reduce_decode()                            # line 12-13
    elif not ok_t and not ok_d:
        v = balanced()                                 # line 15-16 (R-14: follow the algorithm)
    elif ok_t and not ok_d and len(state["pending_lens"]) <= slo["w_max"]:
        v = reduce_prefill()                           # line 18-19
    else:
        v = reduce_decode()                            # line 21-22
    if v == 0:
        return N, 0
    u = N - v
    t_p = ev[v][2]
    t_d = layer_time(_phase_shape(model, [1] * len(state["decode_tokens"]),
                                  [int(math.floor(state["decode_mean_ctx"] + 0.5))] * len(state["decode_tokens"])),
                     P, v, u) * 1e3
    k = max(1, int(math.floor(t_p / t_d + 0.5))) if t_d > 0 else 1   # A9: decode steps per prefill layer
    return u, k


# ------------------------------------------------------------ SM ranges

def sm_ranges(p: int, sigma):
    """SM-range work assignment (§8a SG): prefill = sigma[0:p), decode = sigma[p:N)."""
    return list(sigma[:p]), list(sigma[p:])


def default_params(M=148, C_tflops=1649.5, B_gbs=6549.4):
    """Unfitted parameters: d = p = 1 at every m (the plain roofline)."""
    return {
        "M": M, "C_tflops": C_tflops, "B_gbs": B_gbs,
        "d_c": {"m": [1, M], "v": [1.0, 1.0]}, "d_b": {"m": [1, M], "v": [1.0, 1.0]},
        "p_c": 1.0, "p_b": 1.0,
        "tiles": {"gemm_bm": 128, "gemm_bn": 256, "gemm_bk": 64, "min_k_blocks": 4,
                  "attn_bq": 64, "rows_per_unit": 8},
        "occ": {"gemm": 1, "attn": 1, "elem": 4},
    }
