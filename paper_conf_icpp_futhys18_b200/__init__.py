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
                ("wgrad_fused_dy", _c_int), ("dgrad_halo", _c_int),
                ("s_slot_rows", ctypes.c_longlong), ("s_rows_per_sample", ctypes.c_longlong),
                ("wgrad_reduce_wide", _c_int), ("fp32_split", _c_int), ("dgrad_s2d", _c_int)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class DeviceLimits(ctypes.Structure):
    _fields_ = [("sm_count", _c_int), ("max_threads_per_sm", _c_int), ("max_blocks_per_sm", _c_int),
                ("regs_per_sm", _c_int), ("smem_per_sm", _c_int), ("smem_reserved_per_cta", _c_int),
                ("tmem_cols_per_sm", _c_int), ("max_concurrent_kernels", _c_int)]


class KernelAttr(ctypes.Structure):
    _fields_ = [("threads", _c_int), ("regs", _c_int), ("smem_bytes", _c_int), ("tmem_cols", _c_int)]


class PlanOptions(ctypes.Structure):
    """glp_plan_options_t: alternative kernels / tilings of the same computation (bitwise-equal
    outputs; tests and A/B measurements only)."""
    _fields_ = [("cta_pairs", _c_int), ("wgrad_cta_pairs", _c_int), ("halo_wgrad", _c_int),
                ("halo_fwd", _c_int), ("halo_dgrad", _c_int), ("fused_dy", _c_int),
                ("fused_dy_builders", _c_int), ("max_kblocks_per_stage", _c_int),
                ("wgrad_tile_n", _c_int), ("tile_units", _c_int), ("bn_model", _c_int),
                ("pack_block", _c_int), ("s2d_block", _c_int), ("smem_cap", _c_int), ("pdl", _c_int),
                ("wgrad_leaves", _c_int), ("fp32_split", _c_int)]


def plan_options(**kw) -> PlanOptions:
    """The library defaults (glp_plan_options_default) with the given fields replaced."""
    o = PlanOptions()
    _ck(lib().glp_plan_options_default(ctypes.byref(o)), "glp_plan_options_default")
    names = {f for f, _ in PlanOptions._fields_}
    for k, v in kw.items():
        if k not in names:
            raise ValueError(f"unknown plan option {k!r}")
        setattr(o, k, int(v))
    return o


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
           "glp_pool_conv_bwd", "glp_pool_destroy", "glp_conv_desc_set_groups", "glp_sum2",
           "glp_plan_ex", "glp_plan_options_default", "glp_pool_set_launch_term", "glp_pool_get_eq7",
           "glp_tree_sum", "glp_tree_exchange", "glp_stage_reduce_leaves"]

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
        L.glp_plan_ex.argtypes = [P(_vp), _vp, _c_int, _c_int, _c_int, P(PlanOptions)]
        L.glp_plan_options_default.argtypes = [P(PlanOptions)]
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
        L.glp_pool_set_launch_term.argtypes = [_vp, _dbl, _dbl]
        L.glp_pool_get_eq7.argtypes = [_vp, P(_c_int), P(_c_int)]
        L.glp_conv_desc_set_groups.argtypes = [_vp, _c_int]
        L.glp_sum2.argtypes = [_vp, _vp, _vp, _c_size, _vp]
        L.glp_tree_sum.argtypes = [_vp, _c_int, _vp, _c_size, _c_int, _vp]
        L.glp_tree_exchange.argtypes = [_vp, _vp, _c_int, _c_int, _c_size, _vp]
        L.glp_stage_reduce_leaves.argtypes = [_vp, _vp, _vp, _c_size, _vp, _c_size, _vp]
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


def _checked(t, shape, device, name, nullable=False):
    """Pointer of a tensor the kernels will read or write: fp32, contiguous, on the plan's CUDA
    device, exactly `shape` (the kernels index N*C*H*W floats from the pointer, so anything else
    would read or write past the allocation).  Raises ValueError before any library call."""
    if t is None:
        if nullable:
            return None
        raise ValueError(f"{name}: tensor required")
    import torch
    if t.dtype != torch.float32:
        raise ValueError(f"{name}: dtype {t.dtype}, expected torch.float32")
    if not t.is_cuda or t.device.index != device:
        raise ValueError(f"{name}: on {t.device}, expected cuda:{device}")
    if not t.is_contiguous():
        raise ValueError(f"{name}: not contiguous")
    if tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name}: shape {tuple(t.shape)}, expected {tuple(shape)}")
    return ctypes.c_void_p(t.data_ptr())


def _ptrs(ts):
    """Pointer array (const float *const *) of a list of tensors (None entries -> NULL); the
    array object must stay alive for the duration of the call."""
    if ts is None:
        return None
    arr = (ctypes.c_void_p * len(ts))(*[(None if t is None else t.data_ptr()) for t in ts])
    return ctypes.cast(arr, ctypes.c_void_p), arr


def _checked_list(ts, shapes, device, name, nullable=False, entries_nullable=False):
    """Pointer array of per-branch tensors, each checked as _checked (None entries allowed only
    where the library allows them, e.g. a branch without bias)."""
    if ts is None:
        if nullable:
            return None
        raise ValueError(f"{name}: list required")
    if len(ts) != len(shapes):
        raise ValueError(f"{name}: {len(ts)} tensors for {len(shapes)} branches")
    for i, (t, sh) in enumerate(zip(ts, shapes)):
        _checked(t, sh, device, f"{name}[{i}]", nullable=entries_nullable)
    return _ptrs(ts)


def torch_float32():
    import torch
    return torch.float32


def _stream(stream):
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def sum2(a, b, out, stream=None):
    """out = a + b (fp32 CUDA tensors of equal size): the deterministic tree's add (glp_sum2)."""
    dev = a.device.index if a.is_cuda else -1
    pa, pb, po = (_checked(t, tuple(a.shape), dev, n) for t, n in ((a, "a"), (b, "b"), (out, "out")))
    _ck(lib().glp_sum2(pa, pb, po, a.numel(), _stream(stream)), "glp_sum2")
    return out


def _addr_array(addrs):
    arr = (ctypes.c_void_p * len(addrs))(*[int(a) for a in addrs])
    return ctypes.cast(arr, ctypes.c_void_p), arr


def tree_sum(parts, out, accumulate=False, stream=None):
    """out (+)= the fixed balanced binary tree over 1, 2, 4 or 8 equal fp32 CUDA tensors
    (glp_tree_sum): bitwise the dist.tree_sum of glp_sum2 adds, in one launch."""
    dev = out.device.index
    for k, p in enumerate(parts):
        _checked(p, tuple(out.shape), dev, f"parts[{k}]")
    po = _checked(out, tuple(out.shape), dev, "out")
    pa, _keep = _addr_array([p.data_ptr() for p in parts])
    _ck(lib().glp_tree_sum(pa, len(parts), po, out.numel(), int(bool(accumulate)), _stream(stream)),
        "glp_tree_sum")
    return out


def tree_exchange(subtree_ptrs, out_ptrs, rank, count, stream=None):
    """glp_tree_exchange over peer device addresses (ints, e.g. torch symmetric-memory
    buffer_ptrs): this rank's slice of the top tree, stored into every rank's output."""
    ps, _a = _addr_array(subtree_ptrs)
    po, _b = _addr_array(out_ptrs)
    _ck(lib().glp_tree_exchange(ps, po, len(subtree_ptrs), int(rank), int(count), _stream(stream)),
        "glp_tree_exchange")


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
                 samples_in_flight=0, Kw=None, stride_w=None, pad_w=None, branches=None, groups=1,
                 options=None):
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
        opts = options if isinstance(options, PlanOptions) or options is None \
            else plan_options(**options)
        _ck(L.glp_plan_ex(ctypes.byref(self._plan), self._desc, self.device, self.math,
                          int(samples_in_flight), None if opts is None else ctypes.byref(opts)),
            "glp_plan_ex")
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
    # tensor checks (shape, dtype, device, contiguity) before any library call
    def _x(self, t, name="x"):
        return _checked(t, self.x_shape, self.device, name)

    def _y(self, t, name="y"):
        return _checked(t, self.y_shape, self.device, name)

    def _w(self, t, name="w"):
        return _checked(t, self.w_shape, self.device, name)

    def _b(self, t, name="b"):
        return _checked(t, (self.geom.Co,), self.device, name, nullable=True)

    def fwd(self, x, w, b, y, stream=None):
        _ck(lib().glp_conv_fwd(self._plan, self._x(x), self._w(w), self._b(b), self._y(y),
                               ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_fwd")
        return y

    def bwd_data(self, dy, w, dx, stream=None):
        _ck(lib().glp_conv_bwd_data(self._plan, self._y(dy, "dy"), self._w(w), self._x(dx, "dx"),
                                    ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_bwd_data")
        return dx

    def bwd_filter(self, x, dy, dw, db=None, accumulate=False, stream=None):
        _ck(lib().glp_conv_bwd_filter(self._plan, self._x(x), self._y(dy, "dy"), self._w(dw, "dw"),
                                      self._b(db, "db"), int(bool(accumulate)),
                                      ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_bwd_filter")
        return dw, db

    def bwd(self, x, dy, w, dx, dw, db=None, accumulate=False, stream=None):
        pdx = None if dx is None else self._x(dx, "dx")
        _ck(lib().glp_conv_bwd(self._plan, self._x(x), self._y(dy, "dy"), self._w(w), pdx,
                               self._w(dw, "dw"), self._b(db, "db"), int(bool(accumulate)),
                               ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_bwd")
        return dx, dw, db

    # staged execution (include/glp.h "staged execution"): one C call per kernel group
    def stage_pack(self, what, src, stream=None):
        shape = {GLP_PACK_X: self.x_shape, GLP_PACK_DY: self.y_shape, GLP_PACK_DY_DB: self.y_shape}
        p = _checked(src, shape.get(int(what), self.w_shape), self.device, "src")
        _ck(lib().glp_stage_pack(self._plan, int(what), p, ctypes.c_void_p(self.ws_ptr),
                                 self.ws_bytes, _stream(stream)), "glp_stage_pack")

    def stage_fwd(self, b, y, stream=None):
        _ck(lib().glp_stage_fwd(self._plan, self._b(b), self._y(y), ctypes.c_void_p(self.ws_ptr),
                                self.ws_bytes, _stream(stream)), "glp_stage_fwd")

    def stage_bwd_data(self, dx, stream=None):
        _ck(lib().glp_stage_bwd_data(self._plan, self._x(dx, "dx"), ctypes.c_void_p(self.ws_ptr),
                                     self.ws_bytes, _stream(stream)), "glp_stage_bwd_data")

    def stage_bwd_filter(self, stream=None):
        _ck(lib().glp_stage_bwd_filter(self._plan, ctypes.c_void_p(self.ws_ptr), self.ws_bytes,
                                       _stream(stream)), "glp_stage_bwd_filter")

    def stage_reduce(self, dw, db=None, accumulate=False, stream=None):
        _ck(lib().glp_stage_reduce(self._plan, self._w(dw, "dw"), self._b(db, "db"),
                                   int(bool(accumulate)),
                                   ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_stage_reduce")

    def stage_reduce_leaves(self, dw_flat, db_flat, leaf_stride, stream=None):
        """Leaf plans: leaf l's dW / db at dw_flat / db_flat + l * leaf_stride floats (views into
        an [L, stride] leaf buffer; glp_stage_reduce_leaves)."""
        for t, nm in ((dw_flat, "dw"), (db_flat, "db")):
            if t is not None and (t.dtype != torch_float32() or not t.is_cuda or
                                  t.device.index != self.device):
                raise ValueError(f"{nm}: fp32 tensor on cuda:{self.device} required")
        _ck(lib().glp_stage_reduce_leaves(self._plan, _ptr(dw_flat), _ptr(db_flat), int(leaf_stride),
                                          ctypes.c_void_p(self.ws_ptr), self.ws_bytes,
                                          _stream(stream)), "glp_stage_reduce_leaves")

    # fused sibling groups (include/glp.h "fused sibling groups"): one tensor per branch
    def branch_y_shapes(self):
        return [(self.geom.N, c, self.Ho, self.Wo) for c in self.branches]

    def branch_w_shapes(self):
        g = self.geom
        return [(c, g.C, g.Kh, g.Kw) for c in self.branches]

    def _brw(self):
        return self.branch_w_shapes()

    def _bry(self):
        return self.branch_y_shapes()

    def _brb(self):
        return [(c,) for c in self.branches]

    def group_fwd(self, x, ws, bs, ys, stream=None):
        dv = self.device
        (pw, _a) = _checked_list(ws, self._brw(), dv, "w")
        (py, _b) = _checked_list(ys, self._bry(), dv, "y")
        pb = _checked_list(bs, self._brb(), dv, "b", nullable=True, entries_nullable=True)
        _ck(lib().glp_conv_group_fwd(self._plan, self._x(x), pw, None if pb is None else pb[0], py,
                                     ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_group_fwd")
        return ys

    def group_bwd(self, x, dys, ws, dx, dws, dbs=None, accumulate=False, stream=None):
        dv = self.device
        (pdy, _a) = _checked_list(dys, self._bry(), dv, "dy")
        (pw, _b) = _checked_list(ws, self._brw(), dv, "w")
        (pdw, _c) = _checked_list(dws, self._brw(), dv, "dw")
        pdb = _checked_list(dbs, self._brb(), dv, "db", nullable=True)
        pdx = None if dx is None else self._x(dx, "dx")
        _ck(lib().glp_conv_group_bwd(self._plan, self._x(x), pdy, pw, pdx, pdw,
                                     None if pdb is None else pdb[0], int(bool(accumulate)),
                                     ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_conv_group_bwd")
        return dx, dws, dbs

    def stage_pack_group(self, what, srcs, stream=None):
        dv = self.device
        if int(what) == GLP_PACK_X:
            p, _a = _checked_list(srcs, [self.x_shape], dv, "src")
        elif int(what) in (GLP_PACK_DY, GLP_PACK_DY_DB):
            p, _a = _checked_list(srcs, self._bry(), dv, "src")
        else:
            p, _a = _checked_list(srcs, self._brw(), dv, "src")
        _ck(lib().glp_stage_pack_group(self._plan, int(what), p, ctypes.c_void_p(self.ws_ptr),
                                       self.ws_bytes, _stream(stream)), "glp_stage_pack_group")

    def stage_fwd_group(self, bs, ys, stream=None):
        pb = _checked_list(bs, self._brb(), self.device, "b", nullable=True, entries_nullable=True)
        (py, _a) = _checked_list(ys, self._bry(), self.device, "y")
        _ck(lib().glp_stage_fwd_group(self._plan, None if pb is None else pb[0], py,
                                      ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_stage_fwd_group")

    def stage_reduce_group(self, dws, dbs=None, accumulate=False, stream=None):
        (pdw, _a) = _checked_list(dws, self._brw(), self.device, "dw")
        pdb = _checked_list(dbs, self._brb(), self.device, "db", nullable=True)
        _ck(lib().glp_stage_reduce_group(self._plan, pdw, None if pdb is None else pdb[0],
                                         int(bool(accumulate)), ctypes.c_void_p(self.ws_ptr),
                                         self.ws_bytes, _stream(stream)), "glp_stage_reduce_group")

    def debug_im2col(self, x, n, col, stream=None):
        g = self.geom
        pcol = _checked(col, (g.C * g.Kh * g.Kw, self.Ho * self.Wo), self.device, "col")
        _ck(lib().glp_debug_im2col(self._plan, self._x(x), int(n), pcol,
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
        self.device = int(device)
        Ho, Wo = (H + 2 * pad - K) // stride + 1, (W + 2 * pad - K) // stride + 1
        self._shapes = {"x": (N, C, H, W), "y": (N, Co, Ho, Wo), "w": (Co, C, K, K), "b": (Co,)}
        self.eq7_launch_bound = 0
        self.t_kernel_us = self.t_launch_us = None
        self._sync_info()

    def _sync_info(self):
        """Pool size, Eq. 7 bounds and workspace (re-read after a recalibration)."""
        import torch
        L = lib()
        ns, eq7, wsb = _c_int(), _c_int(), _c_size()
        _ck(L.glp_pool_get_info(self._pool, ctypes.byref(ns), ctypes.byref(eq7), ctypes.byref(wsb)),
            "glp_pool_get_info")
        self.n_streams, self.eq7_bound = ns.value, eq7.value
        nbytes = wsb.value + 1024
        if getattr(self, "_ws_nbytes", 0) < nbytes:
            self._ws_buf = torch.empty(nbytes, dtype=torch.uint8, device=f"cuda:{self.device}")
            self._ws_nbytes = nbytes
            off = (-self._ws_buf.data_ptr()) % 1024
            self.ws_ptr = self._ws_buf.data_ptr() + off
            self.ws_bytes = nbytes - off

    def set_launch_term(self, t_kernel_us, t_launch_us):
        """Eq. 7 with the T_K / T_launch term (glp_pool_set_launch_term)."""
        _ck(lib().glp_pool_set_launch_term(self._pool, float(t_kernel_us), float(t_launch_us)),
            "glp_pool_set_launch_term")
        a, b = _c_int(), _c_int()
        _ck(lib().glp_pool_get_eq7(self._pool, ctypes.byref(a), ctypes.byref(b)), "glp_pool_get_eq7")
        self.eq7_launch_bound = b.value
        self.t_kernel_us, self.t_launch_us = float(t_kernel_us), float(t_launch_us)
        self._sync_info()

    def calibrate(self, x, w, b, y):
        """"Profile once" (P173): run the pool's forward once under the CUPTI resource tracker,
        take T_K = the mean duration of the per-sample forward GEMM kernels and T_launch = the
        mean duration of the kernel-launch API calls, and apply Eq. 7's launch term.  Returns
        (T_K us, T_launch us, records of the profiled kernels)."""
        from .tracker import Tracker
        with Tracker() as t:
            self.fwd(x, w, b, y)
        gemm = [k for k in t.kernels if any(s in k.name for s in ("igemm", "hfwd", "simt_fwd"))]
        if not gemm or not t.launch_us:
            raise RuntimeError("resource tracker recorded no forward kernels / launches")
        tk = sum(k.duration_us for k in gemm) / len(gemm)
        tl = sum(t.launch_us) / len(t.launch_us)
        self.set_launch_term(tk, tl)
        return tk, tl, gemm

    def _c(self, t, kind, name, nullable=False):
        return _checked(t, self._shapes[kind], self.device, name, nullable)

    def fwd(self, x, w, b, y, stream=None):
        _ck(lib().glp_pool_conv_fwd(self._pool, self._c(x, "x", "x"), self._c(w, "w", "w"),
                                    self._c(b, "b", "b", True), self._c(y, "y", "y"),
                                    ctypes.c_void_p(self.ws_ptr), self.ws_bytes, _stream(stream)),
            "glp_pool_conv_fwd")
        return y

    def bwd(self, x, dy, w, dx, dw, db=None, stream=None):
        _ck(lib().glp_pool_conv_bwd(self._pool, self._c(x, "x", "x"), self._c(dy, "y", "dy"),
                                    self._c(w, "w", "w"), self._c(dx, "x", "dx", True),
                                    self._c(dw, "w", "dw"), self._c(db, "b", "db", True),
                                    ctypes.c_void_p(self.ws_ptr), self.ws_bytes,
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
