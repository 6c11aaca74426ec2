"""Python binding of libglp.so — the B200-native GLP4NN conv-layer training hot path.

Argument marshalling only: every step of the path runs in the CUDA kernels of ``csrc/``
behind the C ABI of ``include/glp.h`` (same names).  PyTorch supplies device memory and
streams.  There is no CPU fallback: if ``libglp.so`` is missing or no sm_100 device is present
the calls raise.

Paper mapping: glp_conv_fwd = Alg. 1 (P82-99) for a conv layer; glp_conv_bwd_data =
Alg. 2 (P101-121); glp_conv_bwd_filter = the parameter gradients of P129 summed over the
batch; glp_plan = the kernel analyzer + runtime scheduler set-up done once (P167-173).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

PKG = os.path.dirname(os.path.abspath(__file__))
# GLP_LIB overrides the in-tree library (A/B runs of two builds on one box)
LIB_PATH = os.environ.get("GLP_LIB") or os.path.join(PKG, "libglp.so")

# fp32 = 3xTF32 on tcgen05 (fp32-accurate); fp32_simt = the CUDA-core accuracy anchor
GLP_MATH_FP32, GLP_MATH_TF32, GLP_MATH_BF16, GLP_MATH_FP32_SIMT = 0, 1, 2, 3
MATH = {"fp32": GLP_MATH_FP32, "tf32": GLP_MATH_TF32, "bf16": GLP_MATH_BF16,
        "fp32_simt": GLP_MATH_FP32_SIMT}

_c_int, _c_size, _vp, _dbl = ctypes.c_int, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_double


class PlanInfo(ctypes.Structure):
    _fields_ = [("samples_in_flight", _c_int), ("ctas_per_sm", _c_int),
                ("grid_fwd", _c_int), ("grid_bwd_data", _c_int), ("grid_bwd_filter", _c_int),
                ("tile_m", _c_int), ("tile_n_fwd", _c_int), ("tile_n_bwd_data", _c_int),
                ("tile_n_bwd_filter", _c_int), ("stages_fwd", _c_int), ("stages_bwd_data", _c_int),
                ("stages_bwd_filter", _c_int), ("splits_wgrad", _c_int), ("tiles_fwd", _c_int),
                ("tiles_bwd_data", _c_int), ("tiles_bwd_filter", _c_int),
                ("ws_fwd", _c_size), ("ws_bwd_data", _c_size), ("ws_bwd_filter", _c_size),
                ("ws_bwd", _c_size), ("plan_us", _dbl), ("math", _c_int),
                ("wgrad_halo", _c_int), ("fwd_halo", _c_int),
                ("wgrad_fused_dy", _c_int), ("dgrad_halo", _c_int)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class DeviceLimits(ctypes.Structure):
    _fields_ = [("sm_count", _c_int), ("max_threads_per_sm", _c_int), ("max_blocks_per_sm", _c_int),
                ("regs_per_sm", _c_int), ("smem_per_sm", _c_int), ("smem_reserved_per_cta", _c_int),
                ("tmem_cols_per_sm", _c_int), ("max_concurrent_kernels", _c_int)]


class KernelAttr(ctypes.Structure):
    _fields_ = [("threads", _c_int), ("regs", _c_int), ("smem_bytes", _c_int), ("tmem_cols", _c_int)]


# every symbol include/glp.h declares (checked by tests/test_abi.py)
EXPORTS = ["glp_conv_desc_create", "glp_conv_desc_get_output", "glp_conv_desc_destroy", "glp_plan",
           "glp_plan_get_info", "glp_plan_destroy", "glp_conv_fwd", "glp_conv_bwd_data",
           "glp_conv_bwd_filter", "glp_conv_bwd", "glp_device_limits_b200",
           "glp_analyze_ctas_per_sm", "glp_analyze_samples_in_flight", "glp_analyze_eq7",
           "glp_plan_kernel_attr", "glp_status_string", "glp_last_error_string", "glp_version",
           "glp_debug_im2col", "glp_stage_pack", "glp_stage_fwd", "glp_stage_bwd_data",
           "glp_stage_bwd_filter", "glp_stage_reduce", "glp_conv_group_desc_create",
           "glp_conv_group_fwd", "glp_conv_group_bwd", "glp_stage_pack_group", "glp_stage_fwd_group",
           "glp_stage_reduce_group", "glp_pool_create", "glp_pool_get_info", "glp_pool_conv_fwd",
           "glp_pool_conv_bwd", "glp_pool_destroy", "glp_conv_desc_set_groups", "glp_sum2"]

GLP_PACK_X, GLP_PACK_DY, GLP_PACK_DY_DB, GLP_PACK_W_FWD, GLP_PACK_W_BWD_DATA, GLP_PACK_W_BOTH = 0, 1, 2, 3, 4, 5

_lib = None


class GlpError(RuntimeError):
    def __init__(self, status, where):
        L = lib()
        super().__init__(f"{where}: {L.glp_status_string(status).decode()} "
                         f"({L.glp_last_error_string().decode()})")
        self.status = status


def lib():
    """Load libglp.so (fails loudly if it was not built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run __graft_entry__.build() "
                              "(python -m paper_conf_icpp_futhys18_b200._build)")
        L = ctypes.CDLL(LIB_PATH)
        P = ctypes.POINTER
        L.glp_status_string.restype = ctypes.c_char_p
        L.glp_status_string.argtypes = [_c_int]
        L.glp_last_error_string.restype = ctypes.c_char_p
        L.glp_version.restype = _c_int
        L.glp_conv_desc_create.argtypes = [P(_vp)] + [_c_int] * 11
        L.glp_conv_desc_get_output.argtypes = [_vp, P(_c_int), P(_c_int)]
        L.glp_conv_desc_destroy.argtypes = [_vp]
        L.glp_plan.argtypes = [P(_vp), _vp, _c_int, _c_int, _c_int]
        L.glp_plan_get_info.argtypes = [_vp, P(PlanInfo)]
        L.glp_plan_destroy.argtypes = [_vp]
        L.glp_conv_fwd.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _c_size, _vp]
        L.glp_conv_bwd_data.argtypes = [_vp, _vp, _vp, _vp, _vp, _c_size, _vp]
        L.glp_conv_bwd_filter.argtypes = [_vp, _vp, _vp, _vp, _vp, _c_int, _vp, _c_size, _vp]
        L.glp_conv_bwd.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _vp, _c_int, _vp, _c_size, _vp]
        L.glp_device_limits_b200.argtypes = [P(DeviceLimits)]
        L.glp_analyze_ctas_per_sm.argtypes = [P(DeviceLimits), P(KernelAttr), P(_c_int)]
        L.glp_analyze_samples_in_flight.argtypes = [_c_int, _c_int, _c_int, P(_c_int)]
        L.glp_analyze_eq7.argtypes = [P(DeviceLimits), P(KernelAttr), _c_int, _dbl, _dbl, P(_c_int)]
        L.glp_plan_kernel_attr.argtypes = [_vp, _c_int, P(KernelAttr), P(_c_int), P(_c_int)]
        L.glp_debug_im2col.argtypes = [_vp, _vp, _c_int, _vp, _vp, _c_size, _vp]
        L.glp_stage_pack.argtypes = [_vp, _c_int, _vp, _vp, _c_size, _vp]
        L.glp_stage_fwd.argtypes = [_vp, _vp, _vp, _vp, _c_size, _vp]
        L.glp_stage_bwd_data.argtypes = [_vp, _vp, _vp, _c_size, _vp]
        L.glp_stage_bwd_filter.argtypes = [_vp, _vp, _c_size, _vp]
        L.glp_stage_reduce.argtypes = [_vp, _vp, _vp, _c_int, _vp, _c_size, _vp]
        L.glp_conv_group_desc_create.argtypes = [P(_vp)] + [_c_int] * 5 + [_vp] + [_c_int] * 6
        L.glp_conv_group_fwd.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _c_size, _vp]
        L.glp_conv_group_bwd.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _vp, _c_int, _vp, _c_size, _vp]
        L.glp_stage_pack_group.argtypes = [_vp, _c_int, _vp, _vp, _c_size, _vp]
        L.glp_stage_fwd_group.argtypes = [_vp, _vp, _vp, _vp, _c_size, _vp]
        L.glp_stage_reduce_group.argtypes = [_vp, _vp, _vp, _c_int, _vp, _c_size, _vp]
        L.glp_pool_create.argtypes = [P(_vp), _vp, _c_int, _c_int, _c_int]
        L.glp_pool_get_info.argtypes = [_vp, P(_c_int), P(_c_int), P(_c_size)]
        L.glp_pool_conv_fwd.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _c_size, _vp]
        L.glp_pool_conv_bwd.argtypes = [_vp, _vp, _vp, _vp, _vp, _vp, _vp, _vp, _c_size, _vp]
        L.glp_pool_destroy.argtypes = [_vp]
        L.glp_conv_desc_set_groups.argtypes = [_vp, _c_int]
        L.glp_sum2.argtypes = [_vp, _vp, _vp, _c_size, _vp]
        _lib = L
    return _lib


def _ck(status, where):
    if status != 0:
        raise GlpError(status, where)


# ------------------------------------------------------------------ C-ABI wrappers ---------

def glp_device_limits_b200() -> DeviceLimits:
    lim = DeviceLimits()
    _ck(lib().glp_device_limits_b200(ctypes.byref(lim)), "glp_device_limits_b200")
    return lim


def glp_analyze_ctas_per_sm(lim: DeviceLimits, threads, regs, smem_bytes, tmem_cols) -> int:
    out = _c_int()
    ka = KernelAttr(threads, regs, smem_bytes, tmem_cols)
    _ck(lib().glp_analyze_ctas_per_sm(ctypes.byref(lim), ctypes.byref(ka), ctypes.byref(out)),
        "glp_analyze_ctas_per_sm")
    return out.value


def glp_analyze_samples_in_flight(slots, tiles_per_sample, n_local) -> int:
    out = _c_int()
    _ck(lib().glp_analyze_samples_in_flight(slots, tiles_per_sample, n_local, ctypes.byref(out)),
        "glp_analyze_samples_in_flight")
    return out.value


def glp_analyze_eq7(lim, threads, smem_bytes, blocks, t_kernel=0.0, t_launch=0.0) -> int:
    out = _c_int()
    ka = KernelAttr(threads, 0, smem_bytes, 0)
    _ck(lib().glp_analyze_eq7(ctypes.byref(lim), ctypes.byref(ka), blocks, t_kernel, t_launch,
                              ctypes.byref(out)), "glp_analyze_eq7")
    return out.value


def _ptr(t):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _ptrs(ts):
    """Pointer array (const float *const *) of a list of tensors (None entries -> NULL); the
    array object must stay alive for the duration of the call."""
    if ts is None:
        return None
    arr = (ctypes.c_void_p * len(ts))(*[(None if t is None else t.data_ptr()) for t in ts])
    return ctypes.cast(arr, ctypes.c_void_p), arr


def _stream(stream):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def sum2(a, b, out, stream=None):
    """out = a + b (fp32 CUDA tensors of equal size): the deterministic tree's add (glp_sum2)."""
    _ck(lib().glp_sum2(_ptr(a), _ptr(b), _ptr(out), a.numel(), _stream(stream)), "glp_sum2")
    return out


@dataclass
class Geometry:
    N: int
    C: int
    H: int
    W: int
    Co: int
    Kh: int
    Kw: int
    Sh: int = 1
    Sw: int = 1
    Ph: int = 0
    Pw: int = 0


class ConvLayer:
    """One conv layer plan (glp_conv_desc_create + glp_plan) and its workspace.

    All compute methods take CUDA torch tensors (fp32, contiguous NCHW) and enqueue on
    ``stream`` (default: torch's current stream) without synchronising."""

    def __init__(self, N, C, H, W, Co, K, stride=1, pad=0, math="bf16", device=0,
                 samples_in_flight=0, Kw=None, stride_w=None, pad_w=None, branches=None, groups=1):
        import torch
        self.groups = int(groups)
        self.branches = None if branches is None else [int(c) for c in branches]
        if self.branches is not None:
            Co = sum(self.branches)
        self.geom = Geometry(N, C, H, W, Co, K, Kw or K, stride, stride_w or stride, pad,
                             pad if pad_w is None else pad_w)
        g = self.geom
        L = lib()
        self._desc = _vp()
        if self.branches is None:
            _ck(L.glp_conv_desc_create(ctypes.byref(self._desc), g.N, g.C, g.H, g.W, g.Co, g.Kh,
                                       g.Kw, g.Sh, g.Sw, g.Ph, g.Pw), "glp_conv_desc_create")
        else:
            arr = (_c_int * len(self.branches))(*self.branches)
            _ck(L.glp_conv_group_desc_create(ctypes.byref(self._desc), g.N, g.C, g.H, g.W,
                                             len(self.branches), ctypes.cast(arr, _vp), g.Kh, g.Kw,
                                             g.Sh, g.Sw, g.Ph, g.Pw), "glp_conv_group_desc_create")
        if self.groups != 1:
            _ck(L.glp_conv_desc_set_groups(self._desc, self.groups), "glp_conv_desc_set_groups")
        ho, wo = _c_int(), _c_int()
        _ck(L.glp_conv_desc_get_output(self._desc, ctypes.byref(ho), ctypes.byref(wo)),
            "glp_conv_desc_get_output")
        self.Ho, self.Wo = ho.value, wo.value
        self.math = MATH[math] if isinstance(math, str) else int(math)
        self.device = int(device)
        self._plan = _vp()
        _ck(L.glp_plan(ctypes.byref(self._plan), self._desc, self.device, self.math,
                       int(samples_in_flight)), "glp_plan")
        self.info = PlanInfo()
        _ck(L.glp_plan_get_info(self._plan, ctypes.byref(self.info)), "glp_plan_get_info")
        nbytes = max(self.info.ws_fwd, self.info.ws_bwd_data, self.info.ws_bwd_filter,
                     self.info.ws_bwd, 1) + 1024
        self._ws_buf = torch.empty(nbytes, dtype=torch.uint8, device=f"cuda:{self.device}")
        off = (-self._ws_buf.data_ptr()) % 1024
        self.ws_ptr = self._ws_buf.data_ptr() + off
        self.ws_bytes = nbytes - off

    # shapes
    @property
    def x_shape(self):
        g = self.geom
        return (g.N, g.C, g.H, g.W)

    @property
    def y_shape(self):
        g = self.geom
        return (g.N, g.Co, self.Ho, self.Wo)

    @property
    def w_shape(self):
        g = self.geom
        return (g.Co, g.C // self.groups, g.Kh, g.Kw)

    def kernel_attr(self, which):
        a, m, r = KernelAttr(), _c_int(), _c_int()
        _ck(lib().glp_plan_kernel_attr(self._plan, which, ctypes.byref(a), ctypes.byref(m),
                                       ctypes.byref(r)), "glp_plan_kernel_attr")
        return {"threads": a.threads, "regs": a.regs, "smem": a.smem_bytes,
                "tmem_cols": a.tmem_cols, "model": m.value, "runtime": r.value}

    # compute
    def fwd(self, x, w, b, y, stream=None):
        _ck(lib().glp_conv_fwd(self._plan, _ptr(x), _ptr(w), _ptr(b), _ptr(y),
                               ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_fwd")
        return y

    def bwd_data(self, dy, w, dx, stream=None):
        _ck(lib().glp_conv_bwd_data(self._plan, _ptr(dy), _ptr(w), _ptr(dx),
                                    ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_bwd_data")
        return dx

    def bwd_filter(self, x, dy, dw, db=None, accumulate=False, stream=None):
        _ck(lib().glp_conv_bwd_filter(self._plan, _ptr(x), _ptr(dy), _ptr(dw), _ptr(db),
                                      int(bool(accumulate)), ctypes.c_void_p(self.ws_ptr),
                                      self.ws_bytes, _stream(stream)), "glp_conv_bwd_filter")
        return dw, db

    def bwd(self, x, dy, w, dx, dw, db=None, accumulate=False, stream=None):
        _ck(lib().glp_conv_bwd(self._plan, _ptr(x), _ptr(dy), _ptr(w), _ptr(dx), _ptr(dw),
                               _ptr(db), int(bool(accumulate)), ctypes.c_void_p(self.ws_ptr),
                               self.ws_bytes, _stream(stream)), "glp_conv_bwd")
        return dx, dw, db

    # staged execution (include/glp.h "staged execution"): one C call per kernel group
    def stage_pack(self, what, src, stream=None):
        _ck(lib().glp_stage_pack(self._plan, int(what), _ptr(src), ctypes.c_void_p(self.ws_ptr),
                                 self.ws_bytes, _stream(stream)), "glp_stage_pack")

    def stage_fwd(self, b, y, stream=None):
        _ck(lib().glp_stage_fwd(self._plan, _ptr(b), _ptr(y), ctypes.c_void_p(self.ws_ptr),
                                self.ws_bytes, _stream(stream)), "glp_stage_fwd")

    def stage_bwd_data(self, dx, stream=None):
        _ck(lib().glp_stage_bwd_data(self._plan, _ptr(dx), ctypes.c_void_p(self.ws_ptr),
                                     self.ws_bytes, _stream(stream)), "glp_stage_bwd_data")

    def stage_bwd_filter(self, stream=None):
        _ck(lib().glp_stage_bwd_filter(self._plan, ctypes.c_void_p(self.ws_ptr), self.ws_bytes,
                                       _stream(stream)), "glp_stage_bwd_filter")

    def stage_reduce(self, dw, db=None, accumulate=False, stream=None):
        _ck(lib().glp_stage_reduce(self._plan, _ptr(dw), _ptr(db), int(bool(accumulate)),
                                   ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_stage_reduce")

    # fused sibling groups (include/glp.h "fused sibling groups"): one tensor per branch
    def branch_y_shapes(self):
        return [(self.geom.N, c, self.Ho, self.Wo) for c in self.branches]

    def branch_w_shapes(self):
        g = self.geom
        return [(c, g.C, g.Kh, g.Kw) for c in self.branches]

    def group_fwd(self, x, ws, bs, ys, stream=None):
        (pw, _a), (py, _b) = _ptrs(ws), _ptrs(ys)
        pb = _ptrs(bs)
        _ck(lib().glp_conv_group_fwd(self._plan, _ptr(x), pw, None if pb is None else pb[0], py,
                                     ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_group_fwd")
        return ys

    def group_bwd(self, x, dys, ws, dx, dws, dbs=None, accumulate=False, stream=None):
        (pdy, _a), (pw, _b), (pdw, _c) = _ptrs(dys), _ptrs(ws), _ptrs(dws)
        pdb = _ptrs(dbs)
        _ck(lib().glp_conv_group_bwd(self._plan, _ptr(x), pdy, pw, _ptr(dx), pdw,
                                     None if pdb is None else pdb[0], int(bool(accumulate)),
                                     ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_group_bwd")
        return dx, dws, dbs

    def stage_pack_group(self, what, srcs, stream=None):
        p, _a = _ptrs(srcs)
        _ck(lib().glp_stage_pack_group(self._plan, int(what), p, ctypes.c_void_p(self.ws_ptr),
                                       self.ws_bytes, _stream(stream)), "glp_stage_pack_group")

    def stage_fwd_group(self, bs, ys, stream=None):
        pb, (py, _a) = _ptrs(bs), _ptrs(ys)
        _ck(lib().glp_stage_fwd_group(self._plan, None if pb is None else pb[0], py,
                                      ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_stage_fwd_group")

    def stage_reduce_group(self, dws, dbs=None, accumulate=False, stream=None):
        (pdw, _a), pdb = _ptrs(dws), _ptrs(dbs)
        _ck(lib().glp_stage_reduce_group(self._plan, pdw, None if pdb is None else pdb[0],
                                         int(bool(accumulate)), ctypes.c_void_p(self.ws_ptr),
                                         self.ws_bytes, _stream(stream)), "glp_stage_reduce_group")

    def debug_im2col(self, x, n, col, stream=None):
        _ck(lib().glp_debug_im2col(self._plan, _ptr(x), int(n), _ptr(col),
                                   ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_debug_im2col")
        return col

    def __del__(self):
        try:
            L = lib()
            if getattr(self, "_plan", None):
                L.glp_plan_destroy(self._plan)
            if getattr(self, "_desc", None):
                L.glp_conv_desc_destroy(self._desc)
        except Exception:
            pass


class StreamPool:
    """The paper's prior-art scheme as a comparator (include/glp.h "stream pool"): per-sample
    kernels dispatched round-robin over a pool of streams sized by the Eq. 7 bound."""

    def __init__(self, N, C, H, W, Co, K, stride=1, pad=0, math="bf16", device=0, n_streams=0):
        import torch
        L = lib()
        self.geom = Geometry(N, C, H, W, Co, K, K, stride, stride, pad, pad)
        self._desc = _vp()
        _ck(L.glp_conv_desc_create(ctypes.byref(self._desc), N, C, H, W, Co, K, K, stride, stride,
                                   pad, pad), "glp_conv_desc_create")
        self.math = MATH[math] if isinstance(math, str) else int(math)
        self._pool = _vp()
        _ck(L.glp_pool_create(ctypes.byref(self._pool), self._desc, int(device), self.math,
                              int(n_streams)), "glp_pool_create")
        ns, eq7, wsb = _c_int(), _c_int(), _c_size()
        _ck(L.glp_pool_get_info(self._pool, ctypes.byref(ns), ctypes.byref(eq7), ctypes.byref(wsb)),
            "glp_pool_get_info")
        self.n_streams, self.eq7_bound = ns.value, eq7.value
        nbytes = wsb.value + 1024
        self._ws_buf = torch.empty(nbytes, dtype=torch.uint8, device=f"cuda:{int(device)}")
        off = (-self._ws_buf.data_ptr()) % 1024
        self.ws_ptr = self._ws_buf.data_ptr() + off
        self.ws_bytes = nbytes - off

    def fwd(self, x, w, b, y, stream=None):
        _ck(lib().glp_pool_conv_fwd(self._pool, _ptr(x), _ptr(w), _ptr(b), _ptr(y),
                                    ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_pool_conv_fwd")
        return y

    def bwd(self, x, dy, w, dx, dw, db=None, stream=None):
        _ck(lib().glp_pool_conv_bwd(self._pool, _ptr(x), _ptr(dy), _ptr(w), _ptr(dx), _ptr(dw),
                                    _ptr(db), ctypes.c_void_p(self.ws_ptr), self.ws_bytes,
                                    _stream(stream)), "glp_pool_conv_bwd")
        return dx, dw, db

    def __del__(self):
        try:
            L = lib()
            if getattr(self, "_pool", None):
                L.glp_pool_destroy(self._pool)
            if getattr(self, "_desc", None):
                L.glp_conv_desc_destroy(self._desc)
        except Exception:
            pass
