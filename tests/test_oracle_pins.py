"""Pins for the oracle (CPU only): the oracle is checked against things other than itself.

Each test names what fixes the expected value: a hand-computed worked example (golden file),
a library routine (torch fp64), a mathematical identity (adjoint, finite differences,
1x1 conv = matmul, batch sum), or the paper's stated geometry (Table 5, P316).
"""
import json
import os

import numpy as np
import pytest
import torch

import oracle
from glp_workloads import all_layers, gen_custom

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _t(a):
    return torch.from_numpy(np.asarray(a, np.float64))


# ---------------------------------------------------------------- hand cases (golden) ----

@pytest.mark.parametrize("case", json.load(open(os.path.join(GOLD, "hand_cases.json")))["cases"],
                         ids=lambda c: c["name"])
def test_hand_cases(case):
    x = np.array(case["x"], np.float32)
    w = np.array(case["w"], np.float32)
    b = np.array(case["b"], np.float32)
    dy = np.array(case["dy"], np.float32)
    s, p = case["stride"], case["pad"]
    y = oracle.conv_fwd(x, w, b, s, p)
    np.testing.assert_array_equal(y, np.array(case["y"], np.float64))
    dx = oracle.conv_bwd_data(dy, w, x.shape, s, p)
    np.testing.assert_array_equal(dx, np.array(case["dx"], np.float64))
    dw, db = oracle.conv_bwd_filter(x, dy, w.shape, s, p)
    np.testing.assert_array_equal(dw, np.array(case["dw"], np.float64))
    np.testing.assert_array_equal(db, np.array(case["db"], np.float64))


# ---------------------------------------------------------------- Table 5 geometry --------

def test_table5_output_sizes():
    """Table 5 (P334-355) with the floor reading R2 gives the H_o literals of the workload table."""
    for l in all_layers():
        assert oracle.out_dim(l.H, l.K, l.S, l.P) == l.Ho, l.name


# ---------------------------------------------------------------- library cross-check -----

def _check_torch(x, w, b, dy, s, p, tol=1e-12):
    y = oracle.conv_fwd(x, w, b, s, p)
    yt = torch.nn.functional.conv2d(_t(x), _t(w), _t(b), stride=s, padding=p).numpy()
    assert oracle.normwise_err(y, yt) <= tol
    dx = oracle.conv_bwd_data(dy, w, x.shape, s, p)
    dxt = torch.nn.grad.conv2d_input(x.shape, _t(w), _t(dy), stride=s, padding=p).numpy()
    assert oracle.normwise_err(dx, dxt) <= tol
    dw, db = oracle.conv_bwd_filter(x, dy, w.shape, s, p)
    dwt = torch.nn.grad.conv2d_weight(_t(x), w.shape, _t(dy), stride=s, padding=p).numpy()
    assert oracle.normwise_err(dw, dwt) <= tol
    assert oracle.normwise_err(db, dy.astype(np.float64).sum(axis=(0, 2, 3))) <= tol


@pytest.mark.parametrize("layer", all_layers(), ids=lambda l: f"{l.cfg}-{l.name}")
def test_torch_fp64_config_shapes(layer):
    """torch fp64 conv2d / conv2d_input / conv2d_weight (cross-correlation, zero pad, floor
    output size) on every Table 5 shape at a reduced batch."""
    n = 1 if layer.cfg in (4, 7) else 2
    g = layer.groups   # one group's convolution (the groups are independent convolutions)
    d = gen_custom(n, layer.C // g, layer.H, layer.W, layer.Co // g, layer.K, layer.K,
                   1234 + layer.index, Ho=layer.Ho, Wo=layer.Ho)
    _check_torch(d["x"], d["w"], d["b"], d["dy"], layer.S, layer.P)


@pytest.mark.parametrize("geo", [
    # N, C, H, W, Co, K, S, P   (odd strides/pads, non-square, C=1, H_o=1, ragged)
    (3, 1, 9, 7, 5, 3, 2, 1),
    (2, 5, 11, 13, 4, 5, 3, 2),
    (2, 3, 6, 6, 7, 3, 4, 0),
    (1, 4, 5, 5, 3, 5, 1, 0),       # H_o = 1
    (2, 2, 8, 8, 3, 2, 2, 1),       # even kernel
    (2, 6, 4, 9, 2, 1, 1, 0),       # 1x1
    (1, 3, 10, 10, 2, 3, 1, 3),     # pad > (K-1)/2
])
def test_torch_fp64_odd_shapes(geo):
    N, C, H, W, Co, K, S, P = geo
    Ho, Wo = oracle.out_dim(H, K, S, P), oracle.out_dim(W, K, S, P)
    d = gen_custom(N, C, H, W, Co, K, K, 99, Ho=Ho, Wo=Wo)
    _check_torch(d["x"], d["w"], d["b"], d["dy"], S, P)


# ---------------------------------------------------------------- identities ---------------

@pytest.mark.parametrize("geo", [(3, 4, 9, 9, 5, 3, 2, 1), (2, 3, 13, 13, 6, 5, 1, 2),
                                 (2, 2, 12, 12, 3, 11, 4, 0)])
def test_adjoint_identity(geo):
    """<fwd0(x;W), dy> = <x, dgrad(dy;W)> = <W, wgrad(x,dy)> (bias-free forward)."""
    N, C, H, W, Co, K, S, P = geo
    Ho = oracle.out_dim(H, K, S, P)
    d = gen_custom(N, C, H, W, Co, K, K, 7, Ho=Ho, Wo=Ho)
    y = oracle.conv_fwd(d["x"], d["w"], None, S, P)
    dx = oracle.conv_bwd_data(d["dy"], d["w"], d["x"].shape, S, P)
    dw, _ = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, S, P)
    a = float(np.sum(y * d["dy"].astype(np.float64)))
    bb = float(np.sum(d["x"].astype(np.float64) * dx))
    c = float(np.sum(d["w"].astype(np.float64) * dw))
    scale = max(abs(a), 1e-30)
    assert abs(a - bb) / scale < 1e-13 and abs(a - c) / scale < 1e-13


def test_finite_differences_exact():
    """L = <y(x,W), r>; central differences with h = 0.5 on integer data are exact in fp64
    (conv is linear), so dL/dx == dgrad(r) and dL/dW == wgrad(x, r) bit for bit."""
    N, C, H, W, Co, K, S, P = 2, 3, 7, 7, 4, 3, 2, 1
    Ho = oracle.out_dim(H, K, S, P)
    d = gen_custom(N, C, H, W, Co, K, K, 11, exact=True, Ho=Ho, Wo=Ho)
    x, w, r = d["x"], d["w"], d["dy"]
    dx = oracle.conv_bwd_data(r, w, x.shape, S, P)
    dw, _ = oracle.conv_bwd_filter(x, r, w.shape, S, P)
    L = lambda xx, ww: float(np.sum(oracle.conv_fwd(xx, ww, None, S, P) * r.astype(np.float64)))
    rng = np.random.default_rng(0)
    h = np.float32(0.5)
    for _ in range(12):
        idx = tuple(int(rng.integers(0, s)) for s in x.shape)
        xp, xm = x.copy(), x.copy()
        xp[idx] += h
        xm[idx] -= h
        assert (L(xp, w) - L(xm, w)) / (2 * h) == dx[idx]
        jdx = tuple(int(rng.integers(0, s)) for s in w.shape)
        wp, wm = w.copy(), w.copy()
        wp[jdx] += h
        wm[jdx] -= h
        assert (L(x, wp) - L(x, wm)) / (2 * h) == dw[jdx]


def test_1x1_is_matmul():
    """1x1, stride 1, pad 0 conv == per-sample W[Co,C] @ X[C,HW] (numpy matmul)."""
    N, C, H, W, Co = 3, 7, 5, 6, 4
    d = gen_custom(N, C, H, W, Co, 1, 1, 5, Ho=H, Wo=W)
    y = oracle.conv_fwd(d["x"], d["w"], d["b"], 1, 0)
    w2 = d["w"].reshape(Co, C).astype(np.float64)
    for n in range(N):
        ref = w2 @ d["x"][n].reshape(C, H * W).astype(np.float64) + d["b"].astype(np.float64)[:, None]
        assert oracle.normwise_err(y[n].reshape(Co, -1), ref) < 1e-13
    dw, db = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, 1, 0)
    ref = sum(d["dy"][n].reshape(Co, -1).astype(np.float64) @ d["x"][n].reshape(C, -1).astype(np.float64).T
              for n in range(N))
    assert oracle.normwise_err(dw.reshape(Co, C), ref) < 1e-13


def test_batch_sum_invariant():
    """dW(batch) == sum_n dW(sample n), db likewise (north_star: summed over the samples)."""
    N, C, H, W, Co, K, S, P = 4, 3, 9, 9, 5, 3, 1, 1
    d = gen_custom(N, C, H, W, Co, K, K, 3, Ho=9, Wo=9)
    dw, db = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, S, P)
    acc_w, acc_b = np.zeros_like(dw), np.zeros_like(db)
    for n in range(N):
        a, b = oracle.conv_bwd_filter(d["x"][n:n + 1], d["dy"][n:n + 1], d["w"].shape, S, P)
        acc_w += a
        acc_b += b
    assert oracle.normwise_err(dw, acc_w) < 1e-13 and oracle.normwise_err(db, acc_b) < 1e-13


def test_im2col_gemm_equals_direct_conv_and_unfold():
    """The paper's method (im2col -> sgemm -> bias gemm, P173) reaches the direct definition;
    col layout equals torch.nn.functional.unfold (Caffe row order (ci,kh,kw), col order (ho,wo))."""
    N, C, H, W, Co, K, S, P = 2, 3, 11, 11, 4, 5, 2, 2
    Ho = oracle.out_dim(H, K, S, P)
    d = gen_custom(N, C, H, W, Co, K, K, 21, Ho=Ho, Wo=Ho)
    y = oracle.conv_fwd(d["x"], d["w"], d["b"], S, P)
    for n in range(N):
        col = oracle.im2col(d["x"][n], K, K, S, P)
        unf = torch.nn.functional.unfold(torch.from_numpy(d["x"][n:n + 1]), K, padding=P, stride=S)[0].numpy()
        np.testing.assert_array_equal(col, unf)
        yy = d["w"].reshape(Co, -1).astype(np.float64) @ col.astype(np.float64) + d["b"][:, None]
        assert oracle.normwise_err(y[n].reshape(Co, -1), yy) < 1e-13


def test_thread_count_invariance():
    """OpenMP parallelises over outputs only: 1 thread and all threads are bitwise equal."""
    N, C, H, W, Co, K, S, P = 3, 5, 12, 12, 6, 3, 1, 1
    d = gen_custom(N, C, H, W, Co, K, K, 8, Ho=12, Wo=12)
    mt = oracle.max_threads()
    outs = []
    for t in (1, max(mt, 2)):
        oracle.set_threads(t)
        outs.append((oracle.conv_fwd(d["x"], d["w"], d["b"], S, P),
                     oracle.conv_bwd_data(d["dy"], d["w"], d["x"].shape, S, P),
                     *oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, S, P)))
    oracle.set_threads(mt)
    for a, b in zip(*outs):
        np.testing.assert_array_equal(a, b)


def test_absmode_bounds():
    """absmode computes sum|a||b|, which bounds |sum a b| elementwise."""
    N, C, H, W, Co, K, S, P = 2, 3, 8, 8, 4, 3, 1, 1
    d = gen_custom(N, C, H, W, Co, K, K, 4, Ho=8, Wo=8)
    y = oracle.conv_fwd(d["x"], d["w"], d["b"], S, P)
    ya = oracle.conv_fwd(d["x"], d["w"], d["b"], S, P, absmode=True)
    assert np.all(np.abs(y) <= ya + 1e-15)


def test_absmode_exact_on_nonnegative_operands():
    """Pin of the condition scale sum|a||b| (the full-size float bar): on non-negative operands
    |a||b| = ab, so absmode must equal the plain mode BIT FOR BIT (same loops, same order), for
    every pass and for the one-element forms; and it is invariant under operand sign flips."""
    N, C, H, W, Co, K, S, P = 2, 4, 9, 11, 5, 3, 2, 1
    Ho, Wo = oracle.out_dim(H, K, S, P), oracle.out_dim(W, K, S, P)
    d = gen_custom(N, C, H, W, Co, K, K, 31, Ho=Ho, Wo=Wo)
    x, w, dy = np.abs(d["x"]), np.abs(d["w"]), np.abs(d["dy"])
    np.testing.assert_array_equal(oracle.conv_fwd(x, w, None, S, P, absmode=True),
                                  oracle.conv_fwd(x, w, None, S, P))
    np.testing.assert_array_equal(oracle.conv_bwd_data(dy, w, x.shape, S, P, absmode=True),
                                  oracle.conv_bwd_data(dy, w, x.shape, S, P))
    for a, b in zip(oracle.conv_bwd_filter(x, dy, w.shape, S, P, absmode=True),
                    oracle.conv_bwd_filter(x, dy, w.shape, S, P)):
        np.testing.assert_array_equal(a, b)
    for idx in ((0, 0, 0, 0), (1, 4, Ho - 1, Wo - 1), (1, 2, 1, 3)):
        assert oracle.conv_fwd_at(x, w, None, S, P, idx, absmode=True) == \
            oracle.conv_fwd_at(x, w, None, S, P, idx)
    for idx in ((0, 0, 0, 0), (1, 3, H - 1, W - 1), (0, 2, 4, 5)):
        assert oracle.conv_bwd_data_at(dy, w, x.shape, S, P, idx, absmode=True) == \
            oracle.conv_bwd_data_at(dy, w, x.shape, S, P, idx)
    for idx in ((0, 0, 0, 0), (4, 3, 2, 2), (2, 1, 0, 2)):
        # the numpy form sums in another order than the C loop: equal to rounding only
        assert np.isclose(oracle.conv_bwd_filter_at_abs(x, dy, w.shape, S, P, idx),
                          oracle.conv_bwd_filter_at(x, dy, w.shape, S, P, idx), rtol=1e-14, atol=0)
    # signs do not matter to the condition scale
    np.testing.assert_array_equal(oracle.conv_fwd(-d["x"], d["w"], None, S, P, absmode=True),
                                  oracle.conv_fwd(x, w, None, S, P))


def test_conv_db_definition():
    """conv_db (the bias gradient alone, for full-size checks) equals the db of conv_bwd_filter
    bitwise (same definition and loops) and numpy's fp64 sum over (n, ho, wo)."""
    d = gen_custom(3, 4, 9, 9, 6, 3, 3, 32, Ho=9, Wo=9)
    db = oracle.conv_db(d["dy"])
    _, db2 = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, 1, 1)
    np.testing.assert_array_equal(db, db2)
    np.testing.assert_allclose(db, d["dy"].astype(np.float64).sum(axis=(0, 2, 3)), rtol=1e-13,
                               atol=1e-15)


# ---------------------------------------------------------------- rounding step ------------

def _u(s):
    return np.array([int(s, 16)], np.uint32).view(np.float32)


def test_rounding_bit_patterns():
    g = json.load(open(os.path.join(GOLD, "rounding.json")))
    for a, r in g["tf32_rna"]:
        assert oracle.round_tf32_rna(_u(a)).view(np.uint32)[0] == int(r, 16), a
    for a, r in g["bf16_rne"]:
        assert oracle.round_bf16_rne(_u(a)).view(np.uint32)[0] == int(r, 16), a


def test_rounding_error_bounds():
    """|x - rna_tf32(x)| <= 2^-11 |x|, |x - rne_bf16(x)| <= 2^-8 |x| (half-ulp bounds);
    3xTF32: x - hi exact, |x - hi - lo| <= 2^-22 |x|."""
    rng = np.random.default_rng(1)
    x = (rng.standard_normal(200000) * np.exp(rng.uniform(-20, 20, 200000))).astype(np.float32)
    t = oracle.round_tf32_rna(x).astype(np.float64)
    assert np.all(np.abs(x - t) <= 2.0 ** -11 * np.abs(x))
    assert np.all((t.astype(np.float32).view(np.uint32) & 0x1FFF) == 0)
    bf = oracle.round_bf16_rne(x).astype(np.float64)
    assert np.all(np.abs(x - bf) <= 2.0 ** -8 * np.abs(x))
    assert np.all((bf.astype(np.float32).view(np.uint32) & 0xFFFF) == 0)
    hi, lo = oracle.split_3xtf32(x)
    assert np.all((x.astype(np.float64) - hi) == (x - hi).astype(np.float64))
    assert np.all(np.abs(x.astype(np.float64) - hi - lo) <= 2.0 ** -22 * np.abs(x))


def test_split_mixed_bounds():
    """Mixed split (oracle.split_mixed): hi = rna_tf32(x) and x - hi exact in fp32 (as 3xTF32);
    blo = rne_bf16(x - hi) leaves |x - hi - blo| <= 2^-8 |x - hi| <= 2^-19 |x|; bhi = rne_bf16(hi)
    is a bf16 value within 2^-8 of hi; and the three products the MMAs form represent x*y to
    |x y - (hi_x hi_y + bhi_x blo_y + blo_x bhi_y)| <= 2^-17 |x y| (the two cross terms' bf16
    rounding, 2^-8 of a term <= 2^-11 |x y|, plus the dropped lo*lo)."""
    rng = np.random.default_rng(2)
    x = (rng.standard_normal(200000) * np.exp(rng.uniform(-20, 20, 200000))).astype(np.float32)
    y = (rng.standard_normal(200000) * np.exp(rng.uniform(-20, 20, 200000))).astype(np.float32)
    hi, bhi, blo = oracle.split_mixed(x)
    np.testing.assert_array_equal(hi, oracle.round_tf32_rna(x))
    x64 = x.astype(np.float64)
    assert np.all((x64 - hi) == (x - hi).astype(np.float64))
    assert np.all(np.abs(x64 - hi - blo) <= 2.0 ** -8 * np.abs(x64 - hi))
    assert np.all(np.abs(x64 - hi - blo) <= 2.0 ** -19 * np.abs(x64))
    assert np.all((bhi.view(np.uint32) & 0xFFFF) == 0) and np.all((blo.view(np.uint32) & 0xFFFF) == 0)
    assert np.all(np.abs(bhi.astype(np.float64) - hi) <= 2.0 ** -8 * np.abs(hi.astype(np.float64)))
    hy, bhy, bly = oracle.split_mixed(y)
    prod = (hi.astype(np.float64) * hy + bhi.astype(np.float64) * bly + blo.astype(np.float64) * bhy)
    xy = x64 * y.astype(np.float64)
    assert np.all(np.abs(xy - prod) <= 2.0 ** -17 * np.abs(xy))


def test_sampled_wgrad_element_matches_full():
    N, C, H, W, Co, K, S, P = 3, 4, 9, 9, 5, 3, 2, 1
    Ho = oracle.out_dim(H, K, S, P)
    d = gen_custom(N, C, H, W, Co, K, K, 17, Ho=Ho, Wo=Ho)
    dw, _ = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, S, P)
    for idx in [(0, 0, 0, 0), (4, 3, 2, 2), (2, 1, 0, 2), (1, 2, 1, 1)]:
        assert oracle.conv_bwd_filter_at(d["x"], d["dy"], d["w"].shape, S, P, idx) == dw[idx]


@pytest.mark.parametrize("geo", [(3, 4, 9, 9, 5, 3, 2, 1), (2, 3, 13, 11, 6, 5, 1, 2),
                                 (2, 2, 23, 23, 3, 11, 4, 0), (1, 3, 10, 10, 2, 3, 1, 3),
                                 (2, 6, 4, 9, 2, 1, 1, 0)])
def test_single_element_oracle_matches_full(geo):
    """The one-element forms used by the full-size sampled parity tests (conv_fwd_at,
    conv_bwd_data_at, conv_bwd_filter_at and the |a||b| condition scales) equal the whole-tensor
    oracle — itself pinned above by hand cases, torch fp64 and identities — on every element of
    small tensors (stride 1/2/4, pad 0..3, 1x1, 11x11)."""
    N, C, H, W, Co, K, S, P = geo
    Ho, Wo = oracle.out_dim(H, K, S, P), oracle.out_dim(W, K, S, P)
    d = gen_custom(N, C, H, W, Co, K, K, 23, Ho=Ho, Wo=Wo)
    x, w, b, dy = d["x"], d["w"], d["b"], d["dy"]
    y = oracle.conv_fwd(x, w, b, S, P)
    ya = oracle.conv_fwd(x, w, None, S, P, absmode=True)
    dx = oracle.conv_bwd_data(dy, w, x.shape, S, P)
    dxa = oracle.conv_bwd_data(dy, w, x.shape, S, P, absmode=True)
    dw, _ = oracle.conv_bwd_filter(x, dy, w.shape, S, P)
    dwa, _ = oracle.conv_bwd_filter(x, dy, w.shape, S, P, absmode=True)
    for idx in np.ndindex(*y.shape):
        assert oracle.conv_fwd_at(x, w, b, S, P, idx) == pytest.approx(y[idx], rel=1e-12, abs=1e-13)
        assert oracle.conv_fwd_at(x, w, b, S, P, idx, absmode=True) == pytest.approx(ya[idx], rel=1e-12, abs=1e-13)
    for idx in np.ndindex(*x.shape):
        assert oracle.conv_bwd_data_at(dy, w, x.shape, S, P, idx) == pytest.approx(dx[idx], rel=1e-12, abs=1e-13)
        assert oracle.conv_bwd_data_at(dy, w, x.shape, S, P, idx, absmode=True) == pytest.approx(dxa[idx], rel=1e-12, abs=1e-13)
    for idx in np.ndindex(*w.shape):
        assert oracle.conv_bwd_filter_at(x, dy, w.shape, S, P, idx) == pytest.approx(dw[idx], rel=1e-12, abs=1e-13)
        assert oracle.conv_bwd_filter_at_abs(x, dy, w.shape, S, P, idx) == pytest.approx(dwa[idx], rel=1e-12, abs=1e-13)
