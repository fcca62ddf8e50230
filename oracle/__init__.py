"""TEST INFRASTRUCTURE ONLY — the CPU oracle of the Bullet co-run hot path.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_asplos_0001xc0l026_b200`` never imports it, and it
never imports the product: the two share no code.  The only module both sides
use is ``workload.synth`` (seeded input generators, no method arithmetic).

Contents
  bullet_oracle.c   plain fp64 C reference of one decoder layer for a batch of
                    requests with a paged KV pool (prefill and decode alike)
  perfmodel.py      Eq. 1, Eq. 2, T_m and the Alg. 1 split decision, written
                    out plainly, with brute-force split enumeration
  This file         ctypes loader + numpy marshalling for bullet_oracle.c

Every function cites the PAPER.md line ("P:Lnnn") it follows; readings of
passages the paper leaves open are listed in DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bullet_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile bullet_oracle.c into liboracle.so (gcc, OpenMP, no -march)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-D_DEFAULT_SOURCE", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


class _Cfg(ctypes.Structure):
    _fields_ = [("d_model", ctypes.c_int), ("n_heads", ctypes.c_int),
                ("n_kv_heads", ctypes.c_int), ("head_dim", ctypes.c_int),
                ("d_ff", ctypes.c_int), ("rms_eps", ctypes.c_double),
                ("rope_theta", ctypes.c_double), ("rope_llama3", ctypes.c_int),
                ("rope_factor", ctypes.c_double), ("rope_low_freq", ctypes.c_double),
                ("rope_high_freq", ctypes.c_double), ("rope_orig_max_pos", ctypes.c_int),
                ("bf16_mirror", ctypes.c_int)]


class _W(ctypes.Structure):
    _fields_ = [(n, ctypes.c_void_p) for n in
                ("w_qkv", "b_qkv", "w_o", "w_gate_up", "w_down", "g_attn", "g_mlp")]


_dp = ctypes.POINTER(ctypes.c_double)


def lib():
    global _lib
    if _lib is None:
        _lib = ctypes.CDLL(build())
        _lib.orc_set_threads.restype = ctypes.c_int
        _lib.orc_set_threads.argtypes = [ctypes.c_int]
        _lib.orc_round_bf16.restype = ctypes.c_double
        _lib.orc_round_bf16.argtypes = [ctypes.c_double]
        _lib.orc_rmsnorm_row.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
                                         ctypes.c_double, ctypes.c_void_p]
        _lib.orc_linear_row.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                        ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
        _lib.orc_rope_inv_freq.argtypes = [ctypes.POINTER(_Cfg), ctypes.c_void_p]
        _lib.orc_rope_apply.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int,
                                        ctypes.c_void_p]
        _lib.orc_slot_offset.restype = ctypes.c_size_t
        _lib.orc_slot_offset.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_int,
                                         ctypes.c_int, ctypes.c_int, ctypes.c_int]
        _lib.orc_attend_paged.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                          ctypes.c_void_p, ctypes.c_int, ctypes.c_int,
                                          ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                          ctypes.c_void_p]
        _lib.orc_layer_forward.restype = ctypes.c_int
        _lib.orc_layer_forward.argtypes = [ctypes.POINTER(_Cfg), ctypes.POINTER(_W),
                                           ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
                                           ctypes.c_int, ctypes.c_int, ctypes.c_void_p,
                                           ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int,
                                           ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p,
                                           ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
    return _lib


@dataclass
class OracleCfg:
    """Model constants the oracle needs (DESIGN.md §3 readings R-1, R-2)."""
    d_model: int
    n_heads: int
    n_kv_heads: int
    head_dim: int
    d_ff: int
    rms_eps: float = 1e-5
    rope_theta: float = 500000.0
    rope_llama3: int = 1
    rope_factor: float = 8.0
    rope_low_freq: float = 1.0
    rope_high_freq: float = 4.0
    rope_orig_max_pos: int = 8192
    bf16_mirror: int = 1

    def c(self) -> _Cfg:
        return _Cfg(self.d_model, self.n_heads, self.n_kv_heads, self.head_dim, self.d_ff,
                    self.rms_eps, self.rope_theta, self.rope_llama3, self.rope_factor,
                    self.rope_low_freq, self.rope_high_freq, self.rope_orig_max_pos,
                    self.bf16_mirror)


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


def _p(a):
    return None if a is None else a.ctypes.data


# ----------------------------------------------------------------- primitives

def set_threads(n: int) -> int:
    """OpenMP threads for the oracle's loops (timing only; n <= 0: all cores).
    Returns the thread count now in effect."""
    return lib().orc_set_threads(int(n))


def round_bf16(x):
    """Round each value to the nearest bf16, ties to even (DESIGN R-3)."""
    f = lib().orc_round_bf16
    x = np.asarray(x, dtype=np.float64)
    return np.vectorize(f, otypes=[np.float64])(x) if x.size else x.copy()


def rmsnorm(x, g, eps):
    """h = x / sqrt(mean(x^2) + eps) * g, row-wise (Llama RMSNorm, DESIGN R-1)."""
    x = _f64(np.atleast_2d(x)); g = _f32(g)
    h = np.empty_like(x)
    for i in range(x.shape[0]):
        lib().orc_rmsnorm_row(_p(x[i]), _p(g), x.shape[1], eps, _p(h[i]))
    return h


def linear(h, W, b=None):
    """y = h W^T (+ b), W stored [N][K] (fp64 accumulate)."""
    h = _f64(np.atleast_2d(h)); W = _f32(W)
    b = None if b is None else _f32(b)
    N, K = W.shape
    y = np.empty((h.shape[0], N))
    for i in range(h.shape[0]):
        lib().orc_linear_row(_p(h[i]), _p(W), _p(b), K, N, _p(y[i]))
    return y


def rope_inv_freq(cfg: OracleCfg):
    out = np.empty(cfg.head_dim // 2)
    c = cfg.c()
    lib().orc_rope_inv_freq(ctypes.byref(c), _p(out))
    return out


def rope_apply(u, pos, inv_freq):
    """Rotate-half RoPE of one head vector at integer position ``pos``."""
    u = _f64(u).copy(); inv_freq = _f64(inv_freq)
    lib().orc_rope_apply(_p(u), u.shape[0], int(pos), _p(inv_freq))
    return u


def slot_offset(bt_row, p, B, Hkv, hd, kvh):
    bt_row = _i32(bt_row)
    return int(lib().orc_slot_offset(_p(bt_row), int(p), B, Hkv, hd, kvh))


def attend_paged(q, pool_k, pool_v, bt_row, B, kvh, last):
    """Softmax attention of one query head over keys 0..last through the block table."""
    pool_k = _f32(pool_k); pool_v = _f32(pool_v); bt_row = _i32(bt_row); q = _f64(q)
    _, Hkv, _, hd = pool_k.shape
    o = np.empty(hd)
    lib().orc_attend_paged(_p(q), _p(pool_k), _p(pool_v), _p(bt_row), B, Hkv, hd, kvh,
                           int(last), _p(o))
    return o


# ---------------------------------------------------------------- the layer

def layer_forward(cfg: OracleCfg, w: dict, pool_k, pool_v, q_lens, ctx_lens, block_table,
                  x, row_mask=None, diag=False):
    """One decoder layer (DESIGN.md §3 steps 1-9) for requests with ``ctx_lens``
    cached tokens and ``q_lens`` new tokens each.  ``pool_k/pool_v`` (float32,
    [n_blocks][Hkv][B][hd]) are updated in place with the new keys/values.
    Returns fp64 ``out`` [n_rows][d] (rows outside ``row_mask`` are 0), plus a
    dict of diagnostics (q, o, a) when ``diag``."""
    assert pool_k.dtype == np.float32 and pool_k.flags.c_contiguous
    assert pool_v.dtype == np.float32 and pool_v.flags.c_contiguous
    n_blocks, Hkv, B, hd = pool_k.shape
    q_lens = _i32(q_lens); ctx_lens = _i32(ctx_lens); bt = _i32(block_table)
    x = _f64(x)
    n_rows = int(q_lens.sum())
    assert x.shape == (n_rows, cfg.d_model)
    keep = {k: _f32(v) if v is not None else None for k, v in w.items()}
    cw = _W(*[None if keep.get(n) is None else keep[n].ctypes.data for n in
              ("w_qkv", "b_qkv", "w_o", "w_gate_up", "w_down", "g_attn", "g_mlp")])
    mask = None if row_mask is None else np.ascontiguousarray(row_mask, dtype=np.uint8)
    out = np.zeros((n_rows, cfg.d_model))
    qd = od = ad = None
    if diag:
        qd = np.zeros((n_rows, cfg.n_heads * hd)); od = np.zeros_like(qd)
        ad = np.zeros((n_rows, cfg.d_ff))
    c = cfg.c()
    rc = lib().orc_layer_forward(ctypes.byref(c), ctypes.byref(cw), _p(pool_k), _p(pool_v),
                                 n_blocks, B, len(q_lens), _p(q_lens), _p(ctx_lens), _p(bt),
                                 bt.shape[1], _p(x), _p(out), _p(mask), _p(qd), _p(od), _p(ad))
    if rc != 0:
        raise ValueError("orc_layer_forward: invalid arguments")
    if diag:
        return out, {"q": qd, "o": od, "a": ad}
    return out
