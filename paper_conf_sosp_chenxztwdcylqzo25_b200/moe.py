"""Thin ctypes binding of include/moe.h (argument marshalling only).

Every step of the layer runs in libmoe_b200.so; torch is used only to own
device memory and to name the current CUDA stream.  There is no fallback: if
the library is missing this module raises at import time of the binding.
"""
from __future__ import annotations

import ctypes
import os
from typing import Optional

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmoe_b200.so")

MOE_OK = 0
STATUS = {0: "MOE_OK", -1: "MOE_ERR_INVALID_ARG", -2: "MOE_ERR_UNSUPPORTED", -3: "MOE_ERR_OOM",
          -4: "MOE_ERR_CUDA", -5: "MOE_ERR_NCCL", -6: "MOE_ERR_CAPACITY"}
SCORE_SOFTMAX, SCORE_SIGMOID = 0, 1
GROUP_MAX, GROUP_TOP2_SUM = 0, 1
W_BF16, W_FP8, W_F32, W_FP4 = 0, 1, 2, 3

EXPORTED = ["moe_ep_group_forward", "moe_get_unique_id", "moe_layer_create", "moe_layer_forward", "moe_layer_forward_deferred",
            "moe_layer_forward_chained", "moe_tp_group_forward", "moe_layer_destroy", "moe_status_string",
            "moe_last_error", "moe_layer_get_info", "moe_layer_profile", "moe_layer_stage_times", "moe_stage_name",
            "moe_layer_debug_trace"]


class MoEConfig(ctypes.Structure):
    _fields_ = [("hidden", ctypes.c_int32), ("ffn", ctypes.c_int32), ("n_experts", ctypes.c_int32),
                ("top_k", ctypes.c_int32), ("n_group", ctypes.c_int32), ("topk_group", ctypes.c_int32),
                ("group_score", ctypes.c_int32), ("score_fn", ctypes.c_int32), ("norm_topk", ctypes.c_int32),
                ("routed_scale", ctypes.c_float), ("shared_ffn", ctypes.c_int32),
                ("shared_gated", ctypes.c_int32), ("wtype", ctypes.c_int32), ("max_tokens", ctypes.c_int32),
                ("gemv_max_tokens", ctypes.c_int32), ("device", ctypes.c_int32), ("ep_rank", ctypes.c_int32),
                ("ep_size", ctypes.c_int32), ("nccl_unique_id", ctypes.c_void_p), ("tp_rank", ctypes.c_int32),
                ("tp_size", ctypes.c_int32), ("ep_fixed_capacity", ctypes.c_int32)]


class MoEWeights(ctypes.Structure):
    _fields_ = [(n, ctypes.c_void_p) for n in ("gate_w", "gate_bias", "w13", "w13_scale", "w2", "w2_scale",
                                               "ws13", "ws13_scale", "ws2", "ws2_scale", "shared_gate_w")]


class MoERouting(ctypes.Structure):
    _fields_ = [("topk_idx", ctypes.c_void_p), ("topk_w", ctypes.c_void_p),
                ("expert_counts", ctypes.c_void_p), ("perm", ctypes.c_void_p)]


class MoEInfo(ctypes.Structure):
    _fields_ = [("weight_bytes", ctypes.c_int64), ("workspace_bytes", ctypes.c_int64),
                ("gemv_max_tokens", ctypes.c_int32), ("kernels_per_forward_prefill", ctypes.c_int32),
                ("kernels_per_forward_decode", ctypes.c_int32), ("local_experts", ctypes.c_int32)]


_lib = None


def load_library(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libmoe_b200.so (raises if it has not been built -- no fallback)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(f"{path} not built: run `python -m paper_conf_sosp_chenxztwdcylqzo25_b200.build` "
                           "or __graft_entry__.build()")
    lib = ctypes.CDLL(path)
    vp, i32 = ctypes.c_void_p, ctypes.c_int32
    lib.moe_get_unique_id.argtypes = [vp]
    lib.moe_layer_create.argtypes = [ctypes.POINTER(MoEConfig), ctypes.POINTER(MoEWeights), ctypes.POINTER(vp)]
    lib.moe_layer_forward.argtypes = [vp, vp, vp, i32, vp, ctypes.POINTER(MoERouting), vp]
    lib.moe_layer_forward_deferred.argtypes = [vp, vp, vp, i32, i32, vp, vp, vp, ctypes.POINTER(MoERouting), vp]
    lib.moe_layer_forward_chained.argtypes = [vp, vp, vp, i32, i32, vp, vp, vp]
    lib.moe_tp_group_forward.argtypes = [ctypes.POINTER(vp), i32, ctypes.POINTER(vp), ctypes.POINTER(vp), i32, i32,
                                         ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(vp), vp]
    lib.moe_layer_debug_trace.argtypes = [vp, vp, i32]
    lib.moe_layer_destroy.argtypes = [vp]
    lib.moe_status_string.argtypes = [i32]
    lib.moe_status_string.restype = ctypes.c_char_p
    lib.moe_last_error.restype = ctypes.c_char_p
    lib.moe_layer_get_info.argtypes = [vp, ctypes.POINTER(MoEInfo)]
    lib.moe_ep_group_forward.argtypes = [ctypes.POINTER(vp), i32, ctypes.POINTER(vp), ctypes.POINTER(vp),
                                         ctypes.POINTER(i32), i32, ctypes.POINTER(vp), ctypes.POINTER(vp),
                                         ctypes.POINTER(vp), vp]
    lib.moe_ep_group_forward.restype = i32
    lib.moe_layer_profile.argtypes = [vp, i32]
    lib.moe_layer_stage_times.argtypes = [vp, ctypes.POINTER(ctypes.c_float), i32, ctypes.POINTER(i32)]
    lib.moe_stage_name.argtypes = [i32]
    lib.moe_stage_name.restype = ctypes.c_char_p
    for f in ("moe_get_unique_id", "moe_layer_create", "moe_layer_forward", "moe_layer_forward_deferred",
              "moe_layer_forward_chained", "moe_tp_group_forward", "moe_layer_destroy", "moe_layer_get_info",
              "moe_layer_profile", "moe_layer_stage_times", "moe_layer_debug_trace"):
        getattr(lib, f).restype = i32
    _lib = lib
    return lib


class MoEError(RuntimeError):
    def __init__(self, status: int, where: str):
        lib = load_library()
        super().__init__(f"{where}: {STATUS.get(status, status)}: {lib.moe_last_error().decode()}")
        self.status = status


def _check(status: int, where: str):
    if status != MOE_OK:
        raise MoEError(status, where)


def _ptr(t: Optional[torch.Tensor]) -> Optional[int]:
    if t is None:
        return None
    assert t.is_cuda and t.is_contiguous(), "tensors passed to the C ABI must be contiguous CUDA tensors"
    return t.data_ptr()


def get_unique_id() -> bytes:
    lib = load_library()
    buf = ctypes.create_string_buffer(128)
    _check(lib.moe_get_unique_id(buf), "moe_get_unique_id")
    return buf.raw


class MoELayer:
    """One MoE layer handle (moe_layer_create / _forward / _forward_deferred / _destroy)."""

    def __init__(self, preset, weights, max_tokens: int, device: int = 0, gemv_max_tokens: int = 0,
                 ep_rank: int = 0, ep_size: int = 1, unique_id: Optional[bytes] = None, tp_rank: int = 0,
                 tp_size: int = 1, ep_fixed: bool = False):
        lib = load_library()
        self.p = preset
        self.max_tokens = max_tokens
        self.device = device
        self.ep_size = ep_size
        self._uid = ctypes.create_string_buffer(unique_id, 128) if unique_id is not None else None
        cfg = MoEConfig(hidden=preset.hidden, ffn=preset.ffn, n_experts=preset.n_experts, top_k=preset.top_k,
                        n_group=preset.n_group, topk_group=preset.topk_group, group_score=preset.group_score,
                        score_fn=preset.score_fn, norm_topk=int(preset.norm_topk),
                        routed_scale=preset.routed_scale, shared_ffn=preset.shared_ffn,
                        shared_gated=int(preset.shared_gated), wtype=preset.wtype, max_tokens=max_tokens,
                        gemv_max_tokens=gemv_max_tokens, device=device, ep_rank=ep_rank, ep_size=ep_size,
                        nccl_unique_id=ctypes.cast(self._uid, ctypes.c_void_p) if self._uid else None,
                        tp_rank=tp_rank, tp_size=tp_size, ep_fixed_capacity=int(ep_fixed))
        self.tp_size = tp_size
        w = MoEWeights(**{n: _ptr(getattr(weights, n)) for n, _ in MoEWeights._fields_})
        h = ctypes.c_void_p()
        with torch.cuda.device(device):
            _check(lib.moe_layer_create(ctypes.byref(cfg), ctypes.byref(w), ctypes.byref(h)), "moe_layer_create")
        self._h = h
        self._lib = lib

    def info(self) -> MoEInfo:
        inf = MoEInfo()
        _check(self._lib.moe_layer_get_info(self._h, ctypes.byref(inf)), "moe_layer_get_info")
        return inf

    def profile(self, enable: bool = True):
        _check(self._lib.moe_layer_profile(self._h, int(enable)), "moe_layer_profile")

    def stage_times(self) -> dict:
        """Per-stage ms of the last profiled forward (waits for it)."""
        buf = (ctypes.c_float * 32)()
        n = ctypes.c_int32()
        _check(self._lib.moe_layer_stage_times(self._h, buf, 32, ctypes.byref(n)), "moe_layer_stage_times")
        return {self._lib.moe_stage_name(i).decode(): buf[i] for i in range(n.value)}

    def forward(self, x: torch.Tensor, residual: Optional[torch.Tensor] = None, y: Optional[torch.Tensor] = None,
                n_deferred: int = 0, deferred_in: Optional[torch.Tensor] = None,
                deferred_out: Optional[torch.Tensor] = None, want_deferred_out: bool = False,
                routing: Optional[dict] = None, stream: Optional[torch.cuda.Stream] = None):
        """Returns y (and deferred_out when requested).  `routing`, if a dict,
        receives topk_idx / topk_w / expert_counts / perm device tensors."""
        assert x.dtype == torch.bfloat16 and x.dim() == 2 and x.shape[1] == self.p.hidden
        T = x.shape[0]
        if y is None:
            y = torch.empty_like(x)
        if want_deferred_out and deferred_out is None:
            deferred_out = torch.empty_like(x)
        dbg = None
        if routing is not None:
            k = self.p.top_k
            E_loc = self.p.n_experts // self.ep_size
            routing["topk_idx"] = torch.empty((T, k), dtype=torch.int32, device=x.device)
            routing["topk_w"] = torch.empty((T, k), dtype=torch.float32, device=x.device)
            routing["expert_counts"] = torch.empty((E_loc,), dtype=torch.int32, device=x.device)
            routing["perm"] = torch.full((T * k,), -1, dtype=torch.int32, device=x.device)
            dbg = MoERouting(*(routing[n].data_ptr() for n in ("topk_idx", "topk_w", "expert_counts", "perm")))
        st = (stream or torch.cuda.current_stream(x.device)).cuda_stream
        if n_deferred == 0 and deferred_in is None and deferred_out is None:
            s = self._lib.moe_layer_forward(self._h, _ptr(x), _ptr(residual), T, _ptr(y),
                                            ctypes.byref(dbg) if dbg else None, st)
            _check(s, "moe_layer_forward")
            return y
        s = self._lib.moe_layer_forward_deferred(self._h, _ptr(x), _ptr(residual), T, n_deferred,
                                                 _ptr(deferred_in), _ptr(y), _ptr(deferred_out),
                                                 ctypes.byref(dbg) if dbg else None, st)
        _check(s, "moe_layer_forward_deferred")
        return (y, deferred_out) if deferred_out is not None else y

    def forward_chained(self, x: torch.Tensor, residual: Optional[torch.Tensor] = None, n_deferred: int = 0,
                        prev: Optional["MoELayer"] = None, y: Optional[torch.Tensor] = None,
                        stream: Optional[torch.cuda.Stream] = None) -> torch.Tensor:
        """Expert Deferral across layers (include/moe.h moe_layer_forward_chained,
        PAPER.md L241): this layer's last n_deferred slots are left for the next
        layer; `prev`'s deferred slots are computed here and added to y."""
        assert x.dtype == torch.bfloat16 and x.dim() == 2 and x.shape[1] == self.p.hidden
        if y is None:
            y = torch.empty_like(x)
        st = (stream or torch.cuda.current_stream(x.device)).cuda_stream
        s = self._lib.moe_layer_forward_chained(self._h, _ptr(x), _ptr(residual), x.shape[0], n_deferred,
                                                prev._h if prev is not None else None, _ptr(y), st)
        _check(s, "moe_layer_forward_chained")
        return y

    def debug_trace(self, n: int = 4096):
        import numpy as np
        buf = np.zeros(n, dtype=np.uint64)
        _check(self._lib.moe_layer_debug_trace(self._h, buf.ctypes.data, n), "moe_layer_debug_trace")
        return buf

    def close(self):
        if getattr(self, "_h", None):
            self._lib.moe_layer_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def slice_experts(weights, rank: int, ep_size: int):
    """Rank `rank`'s contiguous slice of the routed experts (router and shared
    expert are replicated) -- the weights a rank passes to moe_layer_create."""
    import copy
    E = weights.w13.shape[0]
    n = E // ep_size
    w = copy.copy(weights)
    sl = slice(rank * n, (rank + 1) * n)
    w.w13 = weights.w13[sl].contiguous()
    w.w2 = weights.w2[sl].contiguous()
    if weights.w13_scale is not None:
        w.w13_scale = weights.w13_scale[sl].contiguous()
        w.w2_scale = weights.w2_scale[sl].contiguous()
    return w


def slice_tp(weights, rank: int, tp_size: int, ffn: int, shared_ffn: int):
    """Rank `rank`'s slice for expert tensor parallelism (include/moe.h "Tensor
    parallelism"): 128-column chunks [r n / P, (r+1) n / P) of every expert's FFN
    dimension -- W1 and W3 rows, W2 columns, and their 128x128 block scales."""
    import copy

    def cols(full):
        n = full // 128
        return (rank * n // tp_size) * 128, ((rank + 1) * n // tp_size) * 128

    w = copy.copy(weights)
    c0, c1 = cols(ffn)
    pk = 2 if weights.w2.shape[-1] * 2 == ffn else 1        # FP4: W2 columns are packed 2 per byte
    w.w13 = torch.cat([weights.w13[:, c0:c1], weights.w13[:, ffn + c0:ffn + c1]], dim=1).contiguous()
    w.w2 = weights.w2[:, :, c0 // pk:c1 // pk].contiguous()
    if weights.w13_scale is not None:
        b0, b1, fb = c0 // 128, c1 // 128, ffn // 128
        w.w13_scale = torch.cat([weights.w13_scale[:, b0:b1], weights.w13_scale[:, fb + b0:fb + b1]], dim=1).contiguous()
        w.w2_scale = weights.w2_scale[:, :, b0:b1].contiguous()
    if shared_ffn and weights.ws13 is not None:
        s0, s1 = cols(shared_ffn)
        w.ws13 = torch.cat([weights.ws13[s0:s1], weights.ws13[shared_ffn + s0:shared_ffn + s1]], dim=0).contiguous()
        w.ws2 = weights.ws2[:, s0 // pk:s1 // pk].contiguous()
        if weights.ws13_scale is not None:
            b0, b1, fb = s0 // 128, s1 // 128, shared_ffn // 128
            w.ws13_scale = torch.cat([weights.ws13_scale[b0:b1], weights.ws13_scale[fb + b0:fb + b1]],
                                     dim=0).contiguous()
            w.ws2_scale = weights.ws2_scale[:, b0:b1].contiguous()
    return w


class TPGroup:
    """In-process expert-TP group on one GPU (moe_tp_group_forward): P ranks, each
    holding its 1/P slice of every expert; a forward returns every rank's full y."""

    def __init__(self, preset, weights, tp_size: int, max_tokens: int, device: int = 0):
        self.P = tp_size
        self.layers = [MoELayer(preset, slice_tp(weights, r, tp_size, preset.ffn, preset.shared_ffn),
                                max_tokens=max_tokens, device=device, tp_rank=r, tp_size=tp_size)
                       for r in range(tp_size)]
        self._lib = load_library()

    def forward(self, xs, residuals=None, n_deferred=0, deferred_in=None, want_deferred_out=False, stream=None):
        P = self.P
        vp = ctypes.c_void_p
        arr = lambda ts: (vp * P)(*[None if t is None else _ptr(t) for t in ts]) if ts is not None else None
        ys = [torch.empty_like(x) for x in xs]
        douts = [torch.empty_like(x) for x in xs] if want_deferred_out else None
        st = (stream or torch.cuda.current_stream(xs[0].device)).cuda_stream
        s = self._lib.moe_tp_group_forward((vp * P)(*[l._h.value for l in self.layers]), P, arr(xs), arr(residuals),
                                           xs[0].shape[0], n_deferred, arr(deferred_in), arr(ys), arr(douts), st)
        _check(s, "moe_tp_group_forward")
        return (ys, douts) if want_deferred_out else ys

    def close(self):
        for l in self.layers:
            l.close()


class MoEGroup:
    """In-process expert-parallel group on one GPU (moe_ep_group_forward): P ranks,
    one MoELayer each, owning E/P experts (the NCCL transport runs one process per GPU)."""

    def __init__(self, preset, weights, ep_size: int, max_tokens: int, device: int = 0, ep_fixed: bool = False):
        devices = [device] * ep_size
        self.P = ep_size
        self.layers = []
        for r in range(ep_size):
            wr = slice_experts(weights, r, ep_size)
            if devices[r] != weights.w13.device.index:
                wr = wr.to(f"cuda:{devices[r]}")
            self.layers.append(MoELayer(preset, wr, max_tokens=max_tokens, device=devices[r], ep_rank=r,
                                        ep_size=ep_size, ep_fixed=ep_fixed))
        self._lib = load_library()

    def forward(self, xs, residuals=None, n_deferred=0, deferred_in=None, want_deferred_out=False, stream=None,
                ys=None):
        P = self.P
        vp = ctypes.c_void_p
        arr = lambda ts: (vp * P)(*[None if t is None else _ptr(t) for t in ts]) if ts is not None else None
        ys = ys if ys is not None else [torch.empty_like(x) for x in xs]
        douts = [torch.empty_like(x) for x in xs] if want_deferred_out else None
        T = (ctypes.c_int32 * P)(*[x.shape[0] for x in xs])
        st = (stream or torch.cuda.current_stream(xs[0].device)).cuda_stream
        s = self._lib.moe_ep_group_forward((vp * P)(*[l._h.value for l in self.layers]), P, arr(xs), arr(residuals),
                                           T, n_deferred, arr(deferred_in), arr(ys), arr(douts), st)
        _check(s, "moe_ep_group_forward")
        return (ys, douts) if want_deferred_out else ys

    def close(self):
        for l in self.layers:
            l.close()
