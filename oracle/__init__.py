"""ORACLE — TEST INFRASTRUCTURE ONLY (parity checker, never the product path).

Plain CPU definition of the GLP4NN hot path (Alg. 1 P82-99, Alg. 2 P101-121,
parameter gradients P129; conv kernels im2col/sgemm/gemmk P173) with fp64 accumulation,
in ``oracle/oracle.c``, plus the rounding-step definitions (R12) and the
paper's analytical model (``oracle/analyzer.py``, §3.2 Eqs 1-9).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with
``paper_conf_icpp_futhys18_b200`` and does not import it.

Parity status per function (see DESIGN.md §Oracle pins):
  conv_fwd / conv_bwd_data / conv_bwd_filter / conv_db / im2col -- pinned (hand cases, torch fp64,
      adjoint identity, finite differences, 1x1 = matmul, batch-sum, floor truncation,
      im2col+GEMM == direct conv, thread-count invariance; conv_db == the bwd_filter db bitwise
      and numpy's sum; absmode == the plain mode bitwise on non-negative operands)
  round_tf32_rna / round_bf16_rne / split_3xtf32          -- pinned (bit patterns, error bound)
  analyzer.*                                              -- pinned (paper worked example P173,
      brute-force MILP enumeration vs closed form)
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc -O2 -fopenmp (no CUDA, no shared headers)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        i, p = ctypes.c_int, ctypes.c_void_p
        L.oracle_conv_fwd.argtypes = [i] * 11 + [p, p, p, p, i]
        L.oracle_conv_bwd_data.argtypes = [i] * 11 + [p, p, p, i]
        L.oracle_conv_bwd_filter.argtypes = [i] * 11 + [p, p, p, p, i]
        L.oracle_im2col.argtypes = [i] * 9 + [p, p]
        L.oracle_conv_db.argtypes = [i] * 4 + [p, p]
        L.oracle_conv_bwd_filter_at.argtypes = [i] * 11 + [p, p, i, i, i, i]
        L.oracle_conv_bwd_filter_at.restype = ctypes.c_double
        L.oracle_set_threads.argtypes = [i]
        L.oracle_max_threads.restype = i
        _lib = L
    return _lib


def set_threads(n: int) -> None:
    lib().oracle_set_threads(int(n))


def max_threads() -> int:
    return int(lib().oracle_max_threads())


def out_dim(n: int, k: int, s: int, p: int) -> int:
    """Table 5 (P316) output size, floor reading (R2)."""
    return (n + 2 * p - k) // s + 1


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def _geom(x_shape, w_shape, stride, pad):
    N, C, H, W = x_shape
    Co, Ci, Kh, Kw = w_shape
    assert Ci == C, "group = 1 (DESIGN.md R4)"
    sh, sw = (stride, stride) if np.isscalar(stride) else stride
    ph, pw = (pad, pad) if np.isscalar(pad) else pad
    return N, C, H, W, Co, Kh, Kw, int(sh), int(sw), int(ph), int(pw)


def conv_fwd(x, w, b=None, stride=1, pad=0, absmode=False):
    """Alg. 1 (P82-99): y = b + W (*) x, fp64 result."""
    x, w = _f32(x), _f32(w)
    b = _f32(b) if b is not None else None
    g = _geom(x.shape, w.shape, stride, pad)
    N, C, H, W, Co, Kh, Kw, sh, sw, ph, pw = g
    y = np.empty((N, Co, out_dim(H, Kh, sh, ph), out_dim(W, Kw, sw, pw)), np.float64)
    lib().oracle_conv_fwd(*g, _ptr(x), _ptr(w), _ptr(b), _ptr(y), int(absmode))
    return y


def conv_bwd_data(dy, w, x_shape, stride=1, pad=0, absmode=False):
    """Alg. 2 (P101-121): dx = col2im(W^T dy), fp64 result (scatter-add formulation)."""
    dy, w = _f32(dy), _f32(w)
    g = _geom(x_shape, w.shape, stride, pad)
    dx = np.empty(tuple(x_shape), np.float64)
    lib().oracle_conv_bwd_data(*g, _ptr(dy), _ptr(w), _ptr(dx), int(absmode))
    return dx


def conv_bwd_filter(x, dy, w_shape, stride=1, pad=0, with_bias=True, absmode=False):
    """P129 parameter gradients summed over the batch: (dW, db) in fp64."""
    x, dy = _f32(x), _f32(dy)
    g = _geom(x.shape, w_shape, stride, pad)
    dw = np.empty(tuple(w_shape), np.float64)
    db = np.empty((w_shape[0],), np.float64) if with_bias else None
    lib().oracle_conv_bwd_filter(*g, _ptr(x), _ptr(dy), _ptr(dw), _ptr(db), int(absmode))
    return dw, db


def conv_db(dy):
    """P129 bias gradient alone: db[co] = sum_{n,ho,wo} dy[n,co,ho,wo] (fp64), the same loops as
    conv_bwd_filter's db."""
    dy = _f32(dy)
    N, Co, Ho, Wo = dy.shape
    db = np.empty((Co,), np.float64)
    lib().oracle_conv_db(N, Co, Ho, Wo, _ptr(dy), _ptr(db))
    return db


def conv_bwd_filter_at(x, dy, w_shape, stride, pad, idx):
    """One dW[co,ci,kh,kw] element (fp64), same definition as conv_bwd_filter."""
    x, dy = _f32(x), _f32(dy)
    g = _geom(x.shape, w_shape, stride, pad)
    co, ci, kh, kw = (int(v) for v in idx)
    return float(lib().oracle_conv_bwd_filter_at(*g, _ptr(x), _ptr(dy), co, ci, kh, kw))


def conv_fwd_at(x, w, b, stride, pad, idx, absmode=False):
    """One y[n,co,ho,wo] (fp64) by the definition of Alg. 1 (P82-99) / SURVEY a3:
    y = b[co] + sum_{ci,kh,kw} W[co,ci,kh,kw] * x[n,ci,ho*S-P+kh, wo*S-P+kw] (zero outside).
    absmode: sum of |W||x| (the element's condition scale; bias excluded).  For sampled parity at
    full size, where the whole-tensor oracle would take too long."""
    n, co, ho, wo = (int(v) for v in idx)
    _, C, H, W = x.shape
    _, _, Kh, Kw = w.shape
    acc = 0.0
    for kh in range(Kh):
        ih = ho * stride - pad + kh
        if ih < 0 or ih >= H:
            continue
        for kw in range(Kw):
            iw = wo * stride - pad + kw
            if iw < 0 or iw >= W:
                continue
            a = x[n, :, ih, iw].astype(np.float64)
            wv = w[co, :, kh, kw].astype(np.float64)
            acc += float(np.abs(a) @ np.abs(wv)) if absmode else float(a @ wv)
    if not absmode and b is not None:
        acc += float(b[co])
    return acc


def conv_bwd_data_at(dy, w, x_shape, stride, pad, idx, absmode=False):
    """One dx[n,ci,h,w] (fp64) by the gather formula of SURVEY a4 (Alg. 2, P101-121):
    dx = sum over (co, kh, kw) with (h+P-kh) and (w+P-kw) divisible by S and the quotients
    (ho, wo) inside the H_o x W_o output of W[co,ci,kh,kw] * dy[n,co,ho,wo]."""
    n, ci, h, ww = (int(v) for v in idx)
    _, Co, Ho, Wo = dy.shape
    _, _, Kh, Kw = w.shape
    acc = 0.0
    for kh in range(Kh):
        th = h + pad - kh
        if th < 0 or th % stride:
            continue
        ho = th // stride
        if ho >= Ho:
            continue
        for kw in range(Kw):
            tw = ww + pad - kw
            if tw < 0 or tw % stride:
                continue
            wo = tw // stride
            if wo >= Wo:
                continue
            a = dy[n, :, ho, wo].astype(np.float64)
            wv = w[:, ci, kh, kw].astype(np.float64)
            acc += float(np.abs(a) @ np.abs(wv)) if absmode else float(a @ wv)
    return acc


def conv_bwd_filter_at_abs(x, dy, w_shape, stride, pad, idx):
    """sum_{n,ho,wo} |dy[n,co,ho,wo]| |x[n,ci,ho*S-P+kh, wo*S-P+kw]|: the condition scale of one
    dW element (the plain definition with absolute values; zero outside the image)."""
    co, ci, kh, kw = (int(v) for v in idx)
    N, C, H, W = x.shape
    _, _, Ho, Wo = dy.shape
    hs = np.arange(Ho) * stride - pad + kh
    ws = np.arange(Wo) * stride - pad + kw
    hv, wv = (hs >= 0) & (hs < H), (ws >= 0) & (ws < W)
    xs = np.abs(x[:, ci][:, hs[hv]][:, :, ws[wv]].astype(np.float64))
    ds = np.abs(dy[:, co][:, hv][:, :, wv].astype(np.float64))
    return float((xs * ds).sum())


def im2col(x_n, kh, kw, stride=1, pad=0):
    """Caffe im2col of one sample (C,H,W) -> col[(ci*Kh+kh)*Kw+kw, ho*Wo+wo] (fp32)."""
    x_n = _f32(x_n)
    C, H, W = x_n.shape
    sh, sw = (stride, stride) if np.isscalar(stride) else stride
    ph, pw = (pad, pad) if np.isscalar(pad) else pad
    Ho, Wo = out_dim(H, kh, sh, ph), out_dim(W, kw, sw, pw)
    col = np.empty((C * kh * kw, Ho * Wo), np.float32)
    lib().oracle_im2col(C, H, W, kh, kw, sh, sw, ph, pw, _ptr(x_n), _ptr(col))
    return col


# ----------------------------------------------------------------------------------------
# Rounding-step definitions (R12: the paper is FP32 SIMT; the tensor-core math
# modes round operands once).  Bit-level definitions, pinned by tests/golden/rounding.json.
# ----------------------------------------------------------------------------------------

def round_tf32_rna(a):
    """Round fp32 to TF32 (10 explicit mantissa bits), nearest, ties AWAY from zero.

    Definition: add half an ulp (0x1000) to the magnitude bits, clear the 13 low bits.
    Inf/NaN pass through unchanged."""
    a = _f32(a)
    u = a.view(np.uint32).copy()
    finite = (u & 0x7F800000) != 0x7F800000
    r = ((u.astype(np.uint64) + 0x1000) & 0xFFFFE000).astype(np.uint32)
    u = np.where(finite, r, u)
    return u.view(np.float32)


def round_bf16_rne(a):
    """Round fp32 to bf16 (7 explicit mantissa bits), nearest, ties to EVEN; returned as fp32."""
    a = _f32(a)
    u = a.view(np.uint32).copy()
    finite = (u & 0x7F800000) != 0x7F800000
    lsb = (u >> 16) & 1
    r = ((u.astype(np.uint64) + 0x7FFF + lsb) & 0xFFFF0000).astype(np.uint32)
    u = np.where(finite, r, u)
    return u.view(np.float32)


def split_3xtf32(a):
    """3xTF32 operand split: hi = rna(a), lo = rna(a - hi) (fp32 subtraction)."""
    a = _f32(a)
    hi = round_tf32_rna(a)
    lo = round_tf32_rna((a - hi).astype(np.float32))
    return hi, lo


def split_mixed(a):
    """Mixed fp32 split (DESIGN.md §7 "1xTF32 + 2xBF16"): hi = rna_tf32(a), bhi = rne_bf16(hi),
    blo = rne_bf16(a - hi) (fp32 subtraction, exact).  The products the MMAs form are hi*hi (tf32),
    bhi*blo' and blo*bhi' (bf16); a product a*b' is then represented to ~2^-18 of |a b'|."""
    a = _f32(a)
    hi = round_tf32_rna(a)
    return hi, round_bf16_rne(hi), round_bf16_rne((a - hi).astype(np.float32))


def normwise_err(got, ref):
    """DESIGN.md R11: max_i |g_i - r_i| / max_i |r_i| (per tensor)."""
    ref = np.asarray(ref, np.float64)
    got = np.asarray(got, np.float64)
    den = float(np.max(np.abs(ref))) if ref.size else 0.0
    num = float(np.max(np.abs(got - ref))) if ref.size else 0.0
    return num / den if den > 0 else num
