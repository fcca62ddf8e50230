"""ctypes binding of libbullet.so (include/bullet.h) — argument marshalling
only: every step of the hot path runs in the library's sm_100a kernels.
PyTorch provides device memory and streams.  There is no CPU fallback: if
the library or a B200 is missing, construction raises."""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np
import torch

from . import build as _build

c_int, c_double, c_float, c_void_p = ctypes.c_int, ctypes.c_double, ctypes.c_float, ctypes.c_void_p
P_i32 = ctypes.POINTER(ctypes.c_int32)
P_f64 = ctypes.POINTER(ctypes.c_double)

CORUN, TIMESLICED, UNGATED, SMID_LOG, PROFILE, UNFUSED, UNFUSED_NORM, DEVICE_SPLIT, CHECK_KV = 0, 1, 2, 4, 8, 16, 32, 64, 128
KERNEL_KINDS = ["plan", "rmsnorm1", "qkv", "rope_kv", "attn", "o_proj", "rmsnorm2", "gate_up",
                "down", "allreduce"]
DTYPE_FP32, DTYPE_BF16 = 0, 1
EPI_F32, EPI_RESID, EPI_SILU = 0, 1, 2
ERRORS = {0: "OK", -1: "EINVAL", -2: "ECUDA", -3: "ENCCL", -4: "ESMRANGE", -5: "EKV",
          -6: "ENOMEM", -7: "EUNSUPPORTED"}


class BulletError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"{ERRORS.get(code, code)}: {msg}")
        self.code = code


class ModelCfg(ctypes.Structure):
    _fields_ = [("n_layers", c_int), ("d_model", c_int), ("n_heads", c_int), ("n_kv_heads", c_int),
                ("head_dim", c_int), ("d_ff", c_int), ("rms_eps", c_float), ("rope_theta", c_double),
                ("rope_llama3", c_int), ("rope_factor", c_float), ("rope_low_freq", c_float),
                ("rope_high_freq", c_float), ("rope_orig_max_pos", c_int), ("max_position", c_int),
                ("qkv_bias", c_int), ("dtype", c_int), ("tp_size", c_int), ("tp_rank", c_int),
                ("max_prefill_tokens", c_int), ("max_decode_tokens", c_int)]


class KvPool(ctypes.Structure):
    _fields_ = [("d_k", ctypes.POINTER(c_void_p)), ("d_v", ctypes.POINTER(c_void_p)),
                ("n_blocks", c_int), ("block_size", c_int)]


class LayerWeights(ctypes.Structure):
    _fields_ = [(n, c_void_p) for n in ("w_qkv", "b_qkv", "w_o", "w_gate_up", "w_down", "g_attn", "g_mlp")]


class CBatch(ctypes.Structure):
    _fields_ = [("n_reqs", c_int), ("n_tokens", c_int), ("max_blocks_per_req", c_int),
                ("d_cu_seqlens", c_void_p), ("d_ctx_lens", c_void_p), ("d_block_table", c_void_p),
                ("h_cu_seqlens", c_void_p), ("h_ctx_lens", c_void_p), ("h_block_table", c_void_p),
                ("d_hidden", c_void_p), ("layer_begin", c_int), ("layer_end", c_int)]


class BatchShape(ctypes.Structure):
    _fields_ = [("n_reqs", c_int), ("q_lens", P_i32), ("ctx_lens", P_i32)]


class SchedState(ctypes.Structure):
    _fields_ = [("layers_done", c_int), ("total_layers", c_int), ("n_prefill", c_int),
                ("prefill_lens", P_i32), ("prefill_waited_ms", P_f64), ("n_pending", c_int),
                ("pending_lens", P_i32), ("pending_waited_ms", P_f64), ("n_decode", c_int),
                ("decode_tokens", P_i32), ("decode_elapsed_ms", P_f64), ("decode_mean_ctx", c_double),
                ("u_k", c_int), ("v_k", c_int)]


class Slo(ctypes.Structure):
    _fields_ = [("ttft_norm_ms_per_tok", c_double), ("tpot_ms", c_double), ("w_max", c_int),
                ("v_min", c_int), ("percentile", c_double), ("objective", c_int)]


_lib = None


def lib():
    """Load (building first if missing or stale) the in-tree libbullet.so."""
    global _lib
    if _lib is None:
        path = os.environ.get("BULLET_LIB") or (_build.build() if _build.stale() else _build.OUT)   # override: A/B experiments
        L = ctypes.CDLL(path, mode=ctypes.RTLD_GLOBAL)
        L.bullet_last_error.restype = ctypes.c_char_p
        for name in ("bullet_create", "bullet_perf_create", "bullet_set_layer_weights", "bullet_num_sms", "bullet_sm_order",
                     "bullet_step", "bullet_step_ranges", "bullet_model_predict", "bullet_choose_split",
                     "bullet_set_smid_log", "bullet_sync", "bullet_nccl_unique_id", "bullet_op_gemm",
                     "bullet_op_rmsnorm", "bullet_op_rope_kv", "bullet_op_attention",
                     "bullet_profile_read", "bullet_launch_count", "bullet_tp_base", "bullet_tp_ipc_handle",
                     "bullet_tp_connect", "bullet_tp_connect_ipc", "bullet_tp_hidden", "bullet_set_split",
                     "bullet_get_colocation", "bullet_set_colocation", "bullet_trace_enable",
                     "bullet_trace_read", "bullet_sm_dies", "bullet_gate_fallbacks", "bullet_get_phase_scale",
                     "bullet_set_phase_scale"):
            getattr(L, name).restype = c_int
        L.bullet_create.argtypes = [ctypes.POINTER(ModelCfg), ctypes.POINTER(KvPool), c_void_p,
                                    ctypes.c_char_p, ctypes.POINTER(c_void_p)]
        L.bullet_perf_create.argtypes = [ctypes.POINTER(ModelCfg), c_int, ctypes.c_char_p,
                                         ctypes.POINTER(c_void_p)]
        L.bullet_set_layer_weights.argtypes = [c_void_p, c_int, ctypes.POINTER(LayerWeights)]
        L.bullet_num_sms.argtypes = [c_void_p, ctypes.POINTER(c_int), ctypes.POINTER(c_int)]
        L.bullet_sm_order.argtypes = [c_void_p, P_i32, c_int]
        L.bullet_sm_dies.argtypes = [c_void_p, P_i32, c_int]
        L.bullet_gate_fallbacks.argtypes = [c_void_p, ctypes.POINTER(ctypes.c_longlong)]
        L.bullet_step.argtypes = [c_void_p, ctypes.POINTER(CBatch), ctypes.POINTER(CBatch), c_int, c_int,
                                  c_void_p, c_void_p]
        L.bullet_step_ranges.argtypes = [c_void_p, ctypes.POINTER(CBatch), ctypes.POINTER(CBatch), c_int, c_int,
                                         c_int, c_int, c_int, c_void_p, c_void_p]
        L.bullet_model_predict.argtypes = [c_void_p, ctypes.POINTER(BatchShape), c_int, c_int, P_f64]
        L.bullet_choose_split.argtypes = [c_void_p, ctypes.POINTER(SchedState), ctypes.POINTER(Slo),
                                          ctypes.POINTER(c_int), ctypes.POINTER(c_int)]
        L.bullet_set_smid_log.argtypes = [c_void_p, c_void_p, c_int]
        L.bullet_sync.argtypes = [c_void_p]
        L.bullet_profile_read.argtypes = [c_void_p, P_i32, P_i32, P_i32, ctypes.POINTER(c_float), c_int,
                                          ctypes.POINTER(c_int)]
        L.bullet_launch_count.argtypes = [c_void_p, ctypes.POINTER(ctypes.c_longlong)]
        L.bullet_trace_enable.argtypes = [c_void_p, c_int]
        L.bullet_trace_read.argtypes = [c_void_p, c_void_p, c_void_p, c_int, ctypes.POINTER(c_int)]
        L.bullet_nccl_unique_id.argtypes = [c_void_p]
        L.bullet_tp_base.argtypes = [c_void_p, ctypes.POINTER(c_void_p)]
        L.bullet_set_split.argtypes = [c_void_p, c_int, c_int, c_int, c_int, c_void_p]
        L.bullet_get_colocation.argtypes = [c_void_p, P_f64, P_f64]
        L.bullet_set_colocation.argtypes = [c_void_p, c_double, c_double]
        L.bullet_get_phase_scale.argtypes = [c_void_p, P_f64, P_f64]
        L.bullet_set_phase_scale.argtypes = [c_void_p, c_double, c_double]
        L.bullet_tp_ipc_handle.argtypes = [c_void_p, c_void_p]
        L.bullet_tp_connect.argtypes = [c_void_p, ctypes.POINTER(c_void_p)]
        L.bullet_tp_connect_ipc.argtypes = [c_void_p, c_void_p]
        L.bullet_tp_hidden.argtypes = [c_void_p, c_int, ctypes.POINTER(c_void_p)]
        L.bullet_destroy.argtypes = [c_void_p]
        L.bullet_destroy.restype = None
        L.bullet_op_gemm.argtypes = [c_void_p, c_int, c_void_p, c_int, c_int, c_void_p, c_int, c_int,
                                     c_void_p, c_void_p, c_void_p, c_int, c_int, c_void_p]
        L.bullet_op_stream.restype = c_int
        L.bullet_op_stream_mc.restype = c_int
        L.bullet_op_stream_mc.argtypes = [c_void_p, c_void_p, ctypes.c_size_t, c_int, c_int, c_void_p]
        L.bullet_op_stream.argtypes = [c_void_p, c_void_p, ctypes.c_size_t, c_int, c_int, c_int, c_void_p]
        L.bullet_op_rmsnorm.argtypes = [c_void_p, c_void_p, c_int, c_void_p, c_void_p, c_int, c_int, c_void_p]
        L.bullet_op_rope_kv.argtypes = [c_void_p, ctypes.POINTER(CBatch), c_int, c_void_p, c_void_p,
                                        c_int, c_int, c_void_p]
        L.bullet_op_attention.argtypes = [c_void_p, ctypes.POINTER(CBatch), c_int, c_void_p, c_void_p,
                                          c_int, c_int, c_int, c_void_p]
        _lib = L
    return _lib


def _check(rc):
    if rc != 0:
        raise BulletError(rc, lib().bullet_last_error().decode())


def _ptr(t):
    return None if t is None else c_void_p(t.data_ptr())


def _stream(s):
    if s is None:
        s = torch.cuda.current_stream()
    return c_void_p(s.cuda_stream)


def nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().bullet_nccl_unique_id(buf))
    return buf.raw


class _DeviceArray:
    """__cuda_array_interface__ view of library-owned device memory (the
    PEER-mode symmetric hidden), so torch.as_tensor can alias it."""

    def __init__(self, ptr: int, shape, typestr="<f4"):
        self.__cuda_array_interface__ = {"data": (ptr, False), "shape": tuple(shape), "typestr": typestr,
                                         "version": 3, "strides": None}


class Batch:
    """One phase's batch: device tensors + host mirrors (int32)."""

    def __init__(self, q_lens, ctx_lens, block_table, hidden: torch.Tensor, layer_begin=0,
                 layer_end=1, device="cuda", validate_blocks=True):
        q_lens = np.asarray(q_lens, dtype=np.int32)
        self.ctx_lens = np.ascontiguousarray(ctx_lens, dtype=np.int32)
        self.cu = np.zeros(len(q_lens) + 1, dtype=np.int32)
        self.cu[1:] = np.cumsum(q_lens)
        self.block_table = np.ascontiguousarray(block_table, dtype=np.int32)
        assert self.block_table.ndim == 2 and self.block_table.shape[0] == len(q_lens)
        assert hidden.dtype == torch.float32 and hidden.is_contiguous()
        assert hidden.shape[0] == int(self.cu[-1])
        self.hidden = hidden
        self.d_cu = torch.from_numpy(self.cu).to(device)
        self.d_ctx = torch.from_numpy(self.ctx_lens).to(device)
        self.d_bt = torch.from_numpy(self.block_table).to(device)
        self.layer_begin, self.layer_end = layer_begin, layer_end
        self.validate_blocks = validate_blocks

    @property
    def n_tokens(self):
        return int(self.cu[-1])

    def c(self) -> CBatch:
        b = CBatch()
        b.n_reqs = len(self.ctx_lens); b.n_tokens = self.n_tokens
        b.max_blocks_per_req = self.block_table.shape[1]
        b.d_cu_seqlens = self.d_cu.data_ptr(); b.d_ctx_lens = self.d_ctx.data_ptr()
        b.d_block_table = self.d_bt.data_ptr()
        b.h_cu_seqlens = self.cu.ctypes.data; b.h_ctx_lens = self.ctx_lens.ctypes.data
        b.h_block_table = self.block_table.ctypes.data if self.validate_blocks else None
        b.d_hidden = self.hidden.data_ptr()
        b.layer_begin, b.layer_end = self.layer_begin, self.layer_end
        return b


@dataclass
class Model:
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
    qkv_bias: int = 0
    dtype: str = "bf16"

    @staticmethod
    def of(shape) -> "Model":
        """From any object with the same attribute names (e.g. workload.synth.ModelShape)."""
        return Model(**{k: getattr(shape, k) for k in Model.__dataclass_fields__})

    @property
    def torch_dtype(self):
        return torch.bfloat16 if self.dtype == "bf16" else torch.float32


class Bullet:
    """Handle around bullet_create: one model (per-GPU shard), its KV pools."""

    def __init__(self, model: Model, pools, max_prefill_tokens: int, max_decode_tokens: int,
                 max_position: int, tp_size=1, tp_rank=0, nccl_uids: bytes | None = None,
                 perf_params_json: str | None = None):
        if not torch.cuda.is_available():
            raise RuntimeError("Bullet needs a CUDA device (B200, sm_100a); no CPU fallback")
        self.model = model
        self.pools = pools  # keep alive
        cfg = ModelCfg(len(pools), model.d_model, model.n_heads, model.n_kv_heads, model.head_dim,
                       model.d_ff, model.rms_eps, model.rope_theta, model.rope_llama3,
                       model.rope_factor, model.rope_low_freq, model.rope_high_freq,
                       model.rope_orig_max_pos, max_position, model.qkv_bias,
                       DTYPE_BF16 if model.dtype == "bf16" else DTYPE_FP32, tp_size, tp_rank,
                       max_prefill_tokens, max_decode_tokens)
        n = len(pools)
        self._kp = (c_void_p * n)(*[k.data_ptr() for k, _ in pools])
        self._vp = (c_void_p * n)(*[v.data_ptr() for _, v in pools])
        k0 = pools[0][0]
        pool = KvPool(self._kp, self._vp, k0.shape[0], k0.shape[2])
        h = c_void_p()
        uids = ctypes.create_string_buffer(nccl_uids, 256) if nccl_uids else None
        _check(lib().bullet_create(ctypes.byref(cfg), ctypes.byref(pool), uids,
                                   perf_params_json.encode() if perf_params_json else None,
                                   ctypes.byref(h)))
        self.h = h
        self.weights = {}
        n_sms, gran = c_int(), c_int()
        _check(lib().bullet_num_sms(h, ctypes.byref(n_sms), ctypes.byref(gran)))
        self.n_sms, self.granularity = n_sms.value, gran.value
        self._log = None

    def close(self):
        if getattr(self, "h", None):
            lib().bullet_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_layer_weights(self, layer: int, w: dict):
        self.weights[layer] = w  # keep alive
        lw = LayerWeights(*[None if w.get(n) is None else w[n].data_ptr() for n in
                            ("w_qkv", "b_qkv", "w_o", "w_gate_up", "w_down", "g_attn", "g_mlp")])
        _check(lib().bullet_set_layer_weights(self.h, layer, ctypes.byref(lw)))

    def sm_order(self):
        out = (ctypes.c_int32 * self.n_sms)()
        _check(lib().bullet_sm_order(self.h, out, self.n_sms))
        return list(out)

    def set_smid_log(self, capacity: int | None):
        if capacity:
            self._log = torch.zeros(1 + 4 * capacity, dtype=torch.int32, device="cuda")
            _check(lib().bullet_set_smid_log(self.h, c_void_p(self._log.data_ptr()), capacity))
        else:
            self._log = None
            _check(lib().bullet_set_smid_log(self.h, None, 0))
        return self._log

    def step(self, prefill: Batch | None, decode: Batch | None, prefill_sm_count: int,
             flags: int = CORUN, s_prefill=None, s_decode=None):
        pb = prefill.c() if prefill else None
        db = decode.c() if decode else None
        _check(lib().bullet_step(self.h, ctypes.byref(pb) if pb else None,
                                 ctypes.byref(db) if db else None, int(prefill_sm_count), int(flags),
                                 _stream(s_prefill), _stream(s_decode)))

    def step_ranges(self, prefill: Batch | None, decode: Batch | None, pre_range, dec_range, flags: int = CORUN,
                    s_prefill=None, s_decode=None):
        """Co-run step on explicit (possibly overlapping) SM ranges of sigma."""
        pb = prefill.c() if prefill else None
        db = decode.c() if decode else None
        _check(lib().bullet_step_ranges(self.h, ctypes.byref(pb) if pb else None,
                                        ctypes.byref(db) if db else None, int(pre_range[0]), int(pre_range[1]),
                                        int(dec_range[0]), int(dec_range[1]), int(flags),
                                        _stream(s_prefill), _stream(s_decode)))

    def sync(self):
        _check(lib().bullet_sync(self.h))

    def set_split(self, pre_range, dec_range, stream=None):
        """Device-resident SM sets for steps / graph replays with DEVICE_SPLIT."""
        _check(lib().bullet_set_split(self.h, int(pre_range[0]), int(pre_range[1]), int(dec_range[0]),
                                      int(dec_range[1]), _stream(stream)))

    # ---- fused tensor-parallel all-reduce over peer memory (PEER mode: tp_size > 1, no nccl_uids)
    def tp_base(self) -> int:
        p = c_void_p()
        _check(lib().bullet_tp_base(self.h, ctypes.byref(p)))
        return p.value

    def tp_ipc_handle(self) -> bytes:
        buf = ctypes.create_string_buffer(64)
        _check(lib().bullet_tp_ipc_handle(self.h, buf))
        return buf.raw

    def tp_connect(self, bases):
        arr = (c_void_p * len(bases))(*bases)
        _check(lib().bullet_tp_connect(self.h, arr))

    def tp_connect_ipc(self, handles: bytes):
        buf = ctypes.create_string_buffer(handles, len(handles))
        _check(lib().bullet_tp_connect_ipc(self.h, buf))

    def tp_hidden(self, phase: int, n_tokens: int) -> torch.Tensor:
        """The phase's symmetric fp32 residual stream [n_tokens][d_model] (a
        view of library memory): PEER-mode batches must use it as `hidden`."""
        p = c_void_p()
        _check(lib().bullet_tp_hidden(self.h, int(phase), ctypes.byref(p)))
        return torch.as_tensor(_DeviceArray(p.value, (n_tokens, self.model.d_model)), device="cuda")

    def profile_read(self, cap=1 << 16):
        """[(kind name, phase, layer, ms)] of launches made with PROFILE since the last read."""
        k = (ctypes.c_int32 * cap)(); p = (ctypes.c_int32 * cap)(); l = (ctypes.c_int32 * cap)()
        ms = (c_float * cap)(); n = c_int()
        _check(lib().bullet_profile_read(self.h, k, p, l, ms, cap, ctypes.byref(n)))
        return [(KERNEL_KINDS[k[i]], p[i], l[i], ms[i]) for i in range(n.value)]

    TRACE_CTAS = 2368   # include/bullet.h BULLET_TRACE_CTAS

    def trace_enable(self, max_launches: int):
        """Per-CTA timestamps of the next `max_launches` launches (diagnostics)."""
        _check(lib().bullet_trace_enable(self.h, int(max_launches)))

    def trace_read(self, cap=256):
        """(records uint64 [n][TRACE_CTAS][16], meta int32 [n][4]) of the traced launches."""
        import numpy as np
        rec = np.zeros((cap, self.TRACE_CTAS, 16), dtype=np.uint64)
        meta = np.zeros((cap, 4), dtype=np.int32)
        n = c_int()
        _check(lib().bullet_trace_read(self.h, rec.ctypes.data, meta.ctypes.data, cap, ctypes.byref(n)))
        return rec[:n.value], meta[:n.value]

    def sm_dies(self):
        """Die (0 / 1, -1 unknown) of each SM of sigma, in sigma order."""
        d = (ctypes.c_int32 * self.n_sms)()
        _check(lib().bullet_sm_dies(self.h, d, self.n_sms))
        return list(d)

    def gate_fallbacks(self) -> int:
        n = ctypes.c_longlong()
        _check(lib().bullet_gate_fallbacks(self.h, ctypes.byref(n)))
        return n.value

    def launch_count(self) -> int:
        n = ctypes.c_longlong()
        _check(lib().bullet_launch_count(self.h, ctypes.byref(n)))
        return n.value

    def colocation(self):
        a, b = c_double(), c_double()
        _check(lib().bullet_get_colocation(self.h, ctypes.byref(a), ctypes.byref(b)))
        return a.value, b.value

    def set_colocation(self, p_c: float, p_b: float):
        _check(lib().bullet_set_colocation(self.h, float(p_c), float(p_b)))

    def phase_scale(self):
        a, b = c_double(), c_double()
        _check(lib().bullet_get_phase_scale(self.h, ctypes.byref(a), ctypes.byref(b)))
        return a.value, b.value

    def set_phase_scale(self, pre: float, dec: float):
        """Online level calibration: predicted prefill / decode layer times x pre / dec."""
        _check(lib().bullet_set_phase_scale(self.h, float(pre), float(dec)))

    def predict_us(self, q_lens, ctx_lens, sm_count, corun_sm_count=0) -> float:
        q = np.ascontiguousarray(q_lens, dtype=np.int32); c = np.ascontiguousarray(ctx_lens, dtype=np.int32)
        s = BatchShape(len(q), q.ctypes.data_as(P_i32), c.ctypes.data_as(P_i32))
        out = c_double()
        _check(lib().bullet_model_predict(self.h, ctypes.byref(s), int(sm_count), int(corun_sm_count),
                                          ctypes.byref(out)))
        return out.value

    def choose_split(self, state: dict, slo: dict):
        arr = {}

        def i32(k):
            arr[k] = np.ascontiguousarray(state[k], dtype=np.int32)
            return arr[k].ctypes.data_as(P_i32)

        def f64(k):
            arr[k] = np.ascontiguousarray(state[k], dtype=np.float64)
            return arr[k].ctypes.data_as(P_f64)
        s = SchedState(state["layers_done"], state["total_layers"], len(state["prefill_lens"]),
                       i32("prefill_lens"), f64("prefill_waited_ms"), len(state["pending_lens"]),
                       i32("pending_lens"), f64("pending_waited_ms"), len(state["decode_tokens"]),
                       i32("decode_tokens"), f64("decode_elapsed_ms"), state["decode_mean_ctx"],
                       state["u_k"], state["v_k"])
        sl = Slo(slo["ttft_norm_ms_per_tok"], slo["tpot_ms"], slo["w_max"], slo["v_min"],
                 slo.get("percentile", 0.9), int(slo.get("objective", 0)))
        p, k = c_int(), c_int()
        _check(lib().bullet_choose_split(self.h, ctypes.byref(s), ctypes.byref(sl), ctypes.byref(p),
                                         ctypes.byref(k)))
        return p.value, k.value

    # ---- op-level entry points (per-kernel parity tests)
    def op_gemm(self, epi, A, B, out, bias=None, resid=None, silu_half=0, lo=0, hi=None, stream=None,
                packed=False):
        M, K = A.shape
        N = B.shape[0] if epi != EPI_SILU else 2 * out.shape[1]
        _check(lib().bullet_op_gemm(self.h, epi | (256 if packed else 0), _ptr(A), M, K, _ptr(B), N,
                                    silu_half, _ptr(bias),
                                    _ptr(resid), _ptr(out), lo, self.n_sms if hi is None else hi,
                                    _stream(stream)))

    def op_stream(self, src, mode=0, lo=0, hi=None, stream=None):
        _check(lib().bullet_op_stream(self.h, _ptr(src), src.numel() * src.element_size(), mode, lo,
                                      self.n_sms if hi is None else hi, _stream(stream)))

    def op_stream_mc(self, src, mc, n_ctas, stream=None):
        _check(lib().bullet_op_stream_mc(self.h, _ptr(src), src.numel() * src.element_size(), int(mc), int(n_ctas),
                                         _stream(stream)))

    def op_rmsnorm(self, x, g, out, lo=0, hi=None, stream=None):
        _check(lib().bullet_op_rmsnorm(self.h, _ptr(x), x.shape[0], _ptr(g), _ptr(out), lo,
                                       self.n_sms if hi is None else hi, _stream(stream)))

    def op_rope_kv(self, batch: Batch, layer, qkv, q, lo=0, hi=None, stream=None):
        b = batch.c()
        _check(lib().bullet_op_rope_kv(self.h, ctypes.byref(b), layer, _ptr(qkv), _ptr(q), lo,
                                       self.n_sms if hi is None else hi, _stream(stream)))

    def op_attention(self, batch: Batch, layer, q, o, kind=0, lo=0, hi=None, stream=None):
        b = batch.c()
        _check(lib().bullet_op_attention(self.h, ctypes.byref(b), layer, _ptr(q), _ptr(o), kind, lo,
                                         self.n_sms if hi is None else hi, _stream(stream)))


def declared_symbols(header=None):
    """Function names declared in include/bullet.h."""
    import re
    header = header or os.path.join(_build.ROOT, "include", "bullet.h")
    src = open(header).read()
    return sorted(set(re.findall(r"^\s*(?:int|void|const char \*)\s*(bullet_\w+)\s*\(", src, re.M)))


class PerfModel(Bullet):
    """Host-only handle (bullet_perf_create): the performance estimator and
    split decision without a GPU.  GPU methods raise EUNSUPPORTED."""

    def __init__(self, model: Model, n_sms: int, perf_params_json: str | None = None):
        self.model = model
        cfg = ModelCfg(1, model.d_model, model.n_heads, model.n_kv_heads, model.head_dim, model.d_ff,
                       model.rms_eps, model.rope_theta, model.rope_llama3, model.rope_factor,
                       model.rope_low_freq, model.rope_high_freq, model.rope_orig_max_pos, 1,
                       model.qkv_bias, DTYPE_BF16 if model.dtype == "bf16" else DTYPE_FP32, 1, 0, 0, 0)
        h = c_void_p()
        _check(lib().bullet_perf_create(ctypes.byref(cfg), int(n_sms),
                                        perf_params_json.encode() if perf_params_json else None,
                                        ctypes.byref(h)))
        self.h = h
        self.n_sms, self.granularity = n_sms, 2
        self.weights = {}
