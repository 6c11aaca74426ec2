"""GPU parity of the CUDA path (through the C ABI) against the fp64 oracle.

Bars: normwise max|g-r|/max|r| <= 1e-5 (GLP_MATH_FP32) and <= 2e-2
(TF32/BF16, BASELINE.json north_star); bit-exact on integer-valued inputs in every math mode;
TF32/BF16 vs a rounding-emulated oracle (oracle run on RNA/RNE-rounded operands) <= 1e-4;
bitwise invariance of every output across samples-in-flight S (convergence invariance, P264).
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import gen_custom

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0")
TOL = {"fp32": 1e-5, "fp32_simt": 1e-5, "tf32": 2e-2, "bf16": 2e-2}
# the operand each tensor-core mode's MMA sees (3xTF32: the hi plane for layout checks)
EMU = {"tf32": oracle.round_tf32_rna, "bf16": oracle.round_bf16_rne, "fp32": oracle.round_tf32_rna}

# name, N, C, H, W, Co, K, S, P  — several M tiles, ragged tails, odd geometry
SHAPES = [
    ("lenet_conv2", 4, 20, 12, 12, 50, 5, 1, 0),
    ("cifar_conv1", 3, 3, 32, 32, 32, 5, 1, 2),
    ("caffenet_conv1_s4", 2, 3, 67, 67, 96, 11, 4, 0),
    ("ragged_s2", 3, 13, 9, 11, 37, 3, 2, 1),
    ("gnet_1x1", 5, 832, 7, 7, 48, 1, 1, 0),
    ("gnet_conv_1", 4, 160, 7, 7, 320, 3, 1, 1),
    ("caffenet_conv3", 2, 256, 13, 13, 384, 3, 1, 1),
    ("c1_k5", 2, 1, 28, 28, 20, 5, 1, 0),
    ("ho1", 2, 4, 5, 5, 3, 5, 1, 0),
    ("pad3", 2, 3, 10, 10, 2, 3, 1, 3),
]


def _run(layer, d, math_dev=DEV):
    t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
    y = torch.full(layer.y_shape, float("nan"), device=DEV)
    dx = torch.full(layer.x_shape, float("nan"), device=DEV)
    dw = torch.full(layer.w_shape, float("nan"), device=DEV)
    db = torch.full((layer.geom.Co,), float("nan"), device=DEV)
    layer.fwd(t["x"], t["w"], t["b"], y)
    layer.bwd_data(t["dy"], t["w"], dx)
    layer.bwd_filter(t["x"], t["dy"], dw, db)
    torch.cuda.synchronize()
    return {"y": y.cpu().numpy(), "dx": dx.cpu().numpy(), "dw": dw.cpu().numpy(), "db": db.cpu().numpy()}


def _oracle(d, S, P, x=None, w=None, dy=None):
    x = d["x"] if x is None else x
    w = d["w"] if w is None else w
    dy = d["dy"] if dy is None else dy
    y = oracle.conv_fwd(x, w, d["b"], S, P)
    dx = oracle.conv_bwd_data(dy, w, x.shape, S, P)
    dw, _ = oracle.conv_bwd_filter(x, dy, w.shape, S, P)
    db = oracle.conv_db(d["dy"])   # db is summed from the unrounded fp32 dy in every mode
    return {"y": y, "dx": dx, "dw": dw, "db": db}


def _data(shape, exact=False, seed=1):
    _, N, C, H, W, Co, K, S, P = shape
    Ho, Wo = oracle.out_dim(H, K, S, P), oracle.out_dim(W, K, S, P)
    return gen_custom(N, C, H, W, Co, K, K, seed, exact=exact, Ho=Ho, Wo=Wo, data_fed=exact and C <= 3)


def _layer(shape, math, S=0, **opts):
    """opts: plan options (glp_plan_options_t fields) selecting alternative kernels / tilings."""
    _, N, C, H, W, Co, K, St, P = shape
    return glp.ConvLayer(N, C, H, W, Co, K, St, P, math=math, samples_in_flight=S,
                         options=opts or None)


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32", "fp32_simt"])
@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: s[0])
def test_parity_random(shape, math):
    d = _data(shape)
    got = _run(_layer(shape, math), d)
    ref = _oracle(d, shape[7], shape[8])
    errs = {k: oracle.normwise_err(got[k], ref[k]) for k in ref}
    assert all(np.isfinite(got[k]).all() for k in got), errs
    assert all(e <= TOL[math] for e in errs.values()), errs


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: s[0])
def test_parity_rounding_emulated(shape, math):
    """Oracle on the operands rounded exactly as the pack step defines (oracle.round_*):
    catches indexing bugs that the 2e-2 tolerance would hide.  fp32: the oracle of the products
    the MMAs form (each pass is linear in each operand, so a sum of oracle calls) -- the mixed
    split's hi*hi + bhi*blo + blo*bhi (oracle.split_mixed) where the plan takes it, else 3xTF32's
    hi*hi + hi*lo + lo*hi (oracle.split_3xtf32) -- at 5e-6."""
    d = _data(shape, seed=5)
    layer = _layer(shape, math)
    got = _run(layer, d)
    S, P = shape[7], shape[8]
    if math == "fp32" and layer.info.fp32_split:   # the mixed split's own products
        ref = _mixed_emulated(d, S, P)
        bar = 5e-6
    elif math == "fp32":
        sp = {k: oracle.split_3xtf32(d[k]) for k in ("x", "w", "dy")}
        parts = [_oracle(d, S, P, x=sp["x"][i], w=sp["w"][j], dy=sp["dy"][i])
                 for i, j in ((0, 0), (0, 1), (1, 0))]
        # dW pairs x with dy: its three products are (hi,hi), (hi,lo), (lo,hi) of (x, dy)
        pw = [_oracle(d, S, P, x=sp["x"][i], dy=sp["dy"][j])["dw"] for i, j in ((0, 0), (0, 1), (1, 0))]
        ref = {k: parts[0][k] + parts[1][k] + parts[2][k] for k in ("y", "dx")}
        ref["y"] -= 2 * d["b"].astype(np.float64)[None, :, None, None]   # bias counted once
        ref["dw"] = pw[0] + pw[1] + pw[2]
        ref["db"] = parts[0]["db"]
        bar = 5e-6   # chunked fp32 accumulation of truncating MMAs
    else:
        r = EMU[math]
        ref = _oracle(d, S, P, x=r(d["x"]), w=r(d["w"]), dy=r(d["dy"]))
        bar = 1e-4
    errs = {k: oracle.normwise_err(got[k], ref[k]) for k in ref}
    assert all(e <= bar for e in errs.values()), errs


# layers whose three passes all take TMA operands (channel pitches % 32, unit stride): the mixed
# fp32 split applies (plan option fp32_split = 1)
MIX_SHAPES = [
    ("gnet_conv_1", 4, 160, 7, 7, 320, 3, 1, 1),            # CTA pairs, ragged M tile
    ("caffenet_conv3", 2, 256, 13, 13, 384, 3, 1, 1),
    ("c96_k5_conv2", 2, 96, 27, 27, 256, 5, 1, 2),          # CaffeNet conv2 geometry, K = 2400
    ("c32_k3_ragged", 3, 32, 11, 13, 64, 3, 1, 1),
    ("c64_1x1", 5, 64, 7, 7, 96, 1, 1, 0),
    ("lenet_conv2", 4, 20, 12, 12, 50, 5, 1, 0),            # channel pitches padded to 32
    ("caffenet_conv1_s4", 2, 3, 67, 67, 96, 11, 4, 0),      # space-to-depth; strided dgrad gather
    ("ragged_s2", 3, 13, 9, 11, 37, 3, 2, 1),               # s2d x' 52 -> 64 channels, ragged
]


def _mixed_emulated(d, S, P):
    """Oracle of exactly the products the mixed split's MMAs form: hi*hi + bhi*blo' + blo*bhi'
    with (hi, bhi, blo) = oracle.split_mixed (each pass linear in each operand)."""
    sp = {k: oracle.split_mixed(d[k]) for k in ("x", "w", "dy")}
    pairs = ((0, 0), (1, 2), (2, 1))
    parts = [_oracle(d, S, P, x=sp["x"][i], w=sp["w"][j], dy=sp["dy"][i]) for i, j in pairs]
    pw = [_oracle(d, S, P, x=sp["x"][i], dy=sp["dy"][j])["dw"] for i, j in pairs]
    ref = {k: parts[0][k] + parts[1][k] + parts[2][k] for k in ("y", "dx")}
    ref["y"] -= 2 * d["b"].astype(np.float64)[None, :, None, None]   # bias counted once
    ref["dw"] = pw[0] + pw[1] + pw[2]
    ref["db"] = parts[0]["db"]
    return ref


@pytest.mark.parametrize("shape", MIX_SHAPES, ids=lambda s: s[0])
def test_fp32_mixed_split(shape):
    """GLP_MATH_FP32 with fp32_split = 1 (tf32 hi*hi + two bf16 cross terms): the plan takes the
    split; bit-exact on integer data; within 1e-5 of the fp64 oracle and 5e-6 of the oracle of
    the split's own products on random data; bitwise invariant across samples in flight."""
    layer = _layer(shape, "fp32", fp32_split=1)
    assert layer.info.fp32_split == 1
    S, P = shape[7], shape[8]
    d = _data(shape, exact=True, seed=91)
    got = _run(layer, d)
    ref = _oracle(d, S, P)
    for k in ref:
        np.testing.assert_array_equal(got[k], ref[k].astype(np.float32), err_msg=k)
    d = _data(shape, seed=92)
    runs = [_run(_layer(shape, "fp32", s_, fp32_split=1), d) for s_ in (0, 1, 0)]
    ref = _oracle(d, S, P)
    emu = _mixed_emulated(d, S, P)
    errs = {k: oracle.normwise_err(runs[0][k], ref[k]) for k in ref}
    eerr = {k: oracle.normwise_err(runs[0][k], emu[k]) for k in emu}
    assert all(e <= TOL["fp32"] for e in errs.values()), errs
    assert all(e <= 5e-6 for e in eerr.values()), eerr
    for r in runs[1:]:
        for k in r:
            np.testing.assert_array_equal(r[k], runs[0][k], err_msg=k)


@pytest.mark.parametrize("shape", MIX_SHAPES[:4], ids=lambda s: s[0])
def test_fp32_3xtf32_on_tma_layers(shape):
    """fp32_split = 0 keeps 3xTF32 on layers the mixed split would take (CTA pairs, TMA operands):
    bit-exact on integers and within 5e-6 of the oracle of its own three products."""
    layer = _layer(shape, "fp32", fp32_split=0)
    assert layer.info.fp32_split == 0
    S, P = shape[7], shape[8]
    d = _data(shape, exact=True, seed=93)
    got = _run(layer, d)
    ref = _oracle(d, S, P)
    for k in ref:
        np.testing.assert_array_equal(got[k], ref[k].astype(np.float32), err_msg=k)
    d = _data(shape, seed=94)
    got = _run(layer, d)
    sp = {k: oracle.split_3xtf32(d[k]) for k in ("x", "w", "dy")}
    parts = [_oracle(d, S, P, x=sp["x"][i], w=sp["w"][j], dy=sp["dy"][i])
             for i, j in ((0, 0), (0, 1), (1, 0))]
    pw = [_oracle(d, S, P, x=sp["x"][i], dy=sp["dy"][j])["dw"] for i, j in ((0, 0), (0, 1), (1, 0))]
    ref = {k: parts[0][k] + parts[1][k] + parts[2][k] for k in ("y", "dx")}
    ref["y"] -= 2 * d["b"].astype(np.float64)[None, :, None, None]
    ref["dw"] = pw[0] + pw[1] + pw[2]
    ref["db"] = parts[0]["db"]
    errs = {k: oracle.normwise_err(got[k], ref[k]) for k in ref}
    assert all(e <= 5e-6 for e in errs.values()), errs


def test_fp32_mixed_split_falls_back():
    """Layers whose channel pitch is not a multiple of 32 (the forward / filter gradient would need
    the cp.async gather) keep 3xTF32 under fp32_split = 1; strided layers take the mixed split
    (forward and filter gradient by TMA on the space-to-depth x', the backward-data by the
    K-major gather); the default (2) takes it for unit-stride layers with >= 2 GFLOP per pass
    (CaffeNet conv1's filter gradient measured slower mixed); fp32_split = 0 selects 3xTF32."""
    assert _layer(SHAPES[7], "fp32", fp32_split=1).info.fp32_split == 0    # C = 1: cp.async gather
    assert _layer(SHAPES[2], "fp32", fp32_split=1).info.fp32_split == 1    # stride 4, s2d
    assert _layer(SHAPES[3], "fp32", fp32_split=1).info.fp32_split == 1    # stride 2, s2d
    assert _layer(SHAPES[2], "fp32").info.fp32_split == 0                  # < 2 GFLOP per pass
    conv1 = ("caffenet_conv1_b32", 32, 3, 227, 227, 96, 11, 4, 0)          # 6.7 GFLOP per pass
    assert _layer(conv1, "fp32").info.fp32_split == 0
    assert _layer(conv1, "fp32", fp32_split=1).info.fp32_split == 1
    assert _layer(MIX_SHAPES[0], "fp32").info.fp32_split == 0                # 0.2 GFLOP per pass
    big = ("caffenet_conv3_b8", 8, 256, 13, 13, 384, 3, 1, 1)                 # 2.4 GFLOP per pass
    assert _layer(big, "fp32").info.fp32_split == 1
    assert _layer(big, "fp32", fp32_split=0).info.fp32_split == 0


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32", "fp32_simt"])
@pytest.mark.parametrize("shape", SHAPES, ids=lambda s: s[0])
def test_exact_integer_bitexact(shape, math):
    """Integer data in [-2,2]: every partial sum is an exact integer < 2^24 in fp32/TF32/BF16,
    so the GPU must equal the oracle bit for bit (pins indexing, padding, stride, layout and
    reduction completeness independently of rounding)."""
    d = _data(shape, exact=True, seed=9)
    got = _run(_layer(shape, math), d)
    ref = _oracle(d, shape[7], shape[8])
    for k in ref:
        np.testing.assert_array_equal(got[k], ref[k].astype(np.float32), err_msg=k)


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32", "fp32_simt"])
@pytest.mark.parametrize("shape", [SHAPES[0], SHAPES[2], SHAPES[5], SHAPES[6]], ids=lambda s: s[0])
def test_samples_in_flight_invariance(shape, math):
    """Convergence invariance (P264): outputs bitwise identical for every S and on rerun."""
    d = _data(shape, seed=3)
    N = shape[1]
    base = _run(_layer(shape, math, S=0), d)
    for S in sorted({1, 2, N}):
        got = _run(_layer(shape, math, S=S), d)
        for k in base:
            np.testing.assert_array_equal(got[k], base[k], err_msg=f"S={S} {k}")
    again = _run(_layer(shape, math, S=0), d)
    for k in base:
        np.testing.assert_array_equal(again[k], base[k])


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
@pytest.mark.parametrize("shape", [SHAPES[1], SHAPES[2], SHAPES[3], SHAPES[6]], ids=lambda s: s[0])
def test_im2col_layout_bitexact(shape, math):
    """glp_debug_im2col (the producer's own gather math on the packed operand) equals the
    oracle's Caffe im2col of the rounded input, bit for bit."""
    _, N, C, H, W, Co, K, S, P = shape
    d = _data(shape, seed=4)
    layer = _layer(shape, math)
    x = torch.from_numpy(d["x"]).to(DEV)
    Ho, Wo = layer.Ho, layer.Wo
    for n in sorted({0, N - 1}):
        col = torch.empty((C * K * K, Ho * Wo), device=DEV)
        layer.debug_im2col(x, n, col)
        torch.cuda.synchronize()
        ref = oracle.im2col(EMU[math](d["x"][n]), K, K, S, P)
        np.testing.assert_array_equal(col.cpu().numpy(), ref)


def test_accumulate_flag():
    shape = SHAPES[0]
    d = _data(shape, exact=True, seed=12)
    layer = _layer(shape, "bf16")
    t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
    dw = torch.ones(layer.w_shape, device=DEV)
    db = torch.ones(layer.geom.Co, device=DEV)
    layer.bwd_filter(t["x"], t["dy"], dw, db, accumulate=True)
    torch.cuda.synchronize()
    rdw, _ = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, shape[7], shape[8])
    np.testing.assert_array_equal(dw.cpu().numpy(), (rdw + 1).astype(np.float32))
    np.testing.assert_array_equal(db.cpu().numpy(), (d["dy"].astype(np.float64).sum((0, 2, 3)) + 1).astype(np.float32))


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
def test_combined_bwd_equals_separate(math):
    shape = SHAPES[5]
    d = _data(shape, seed=8)
    layer = _layer(shape, math)
    sep = _run(layer, d)
    t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
    dx = torch.empty(layer.x_shape, device=DEV)
    dw = torch.empty(layer.w_shape, device=DEV)
    db = torch.empty(layer.geom.Co, device=DEV)
    layer.bwd(t["x"], t["dy"], t["w"], dx, dw, db)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(dx.cpu().numpy(), sep["dx"])
    np.testing.assert_array_equal(dw.cpu().numpy(), sep["dw"])
    np.testing.assert_array_equal(db.cpu().numpy(), sep["db"])


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
def test_analyzer_matches_occupancy_api(math):
    """The re-derived analyzer's CTAs/SM for every shipped kernel (the halo kernels included, where
    a plan picks them) equals the CUDA occupancy API."""
    for shape in SHAPES + [("caffenet_conv1_full", 2, 3, 227, 227, 96, 11, 4, 0),
                           ("caffenet_conv2_b2", 2, 96, 27, 27, 256, 5, 1, 2)]:
        layer = _layer(shape, math)
        for which in range(3):
            a = layer.kernel_attr(which)
            assert a["model"] == a["runtime"] >= 1, (shape[0], which, a)


def test_error_paths_on_device():
    layer = _layer(SHAPES[0], "bf16")
    x = torch.zeros(layer.x_shape, device=DEV)
    y = torch.zeros(layer.y_shape, device=DEV)
    w = torch.zeros(layer.w_shape, device=DEV)
    L = glp.lib()
    import ctypes
    rc = L.glp_conv_fwd(layer._plan, ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(w.data_ptr()),
                        None, ctypes.c_void_p(y.data_ptr()), ctypes.c_void_p(layer.ws_ptr), 16, None)
    assert rc == 4  # GLP_ERR_WORKSPACE_TOO_SMALL
    rc = L.glp_conv_fwd(layer._plan, ctypes.c_void_p(x.data_ptr() + 4), ctypes.c_void_p(w.data_ptr()),
                        None, ctypes.c_void_p(y.data_ptr()), ctypes.c_void_p(layer.ws_ptr),
                        layer.ws_bytes, None)
    assert rc == 1  # misaligned


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
def test_staged_equals_composed(math):
    """Staged calls (pack once, GEMMs, reduce) are bitwise identical to the composed calls."""
    shape = SHAPES[6]
    d = _data(shape, seed=14)
    layer = _layer(shape, math)
    ref = _run(layer, d)
    t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
    y = torch.empty(layer.y_shape, device=DEV)
    dx = torch.empty(layer.x_shape, device=DEV)
    dw = torch.empty(layer.w_shape, device=DEV)
    db = torch.empty(layer.geom.Co, device=DEV)
    layer.stage_pack(glp.GLP_PACK_X, t["x"])
    layer.stage_pack(glp.GLP_PACK_W_FWD, t["w"])
    layer.stage_fwd(t["b"], y)
    layer.stage_pack(glp.GLP_PACK_DY_DB, t["dy"])
    layer.stage_pack(glp.GLP_PACK_W_BWD_DATA, t["w"])
    layer.stage_bwd_data(dx)
    layer.stage_bwd_filter()
    layer.stage_reduce(dw, db)
    torch.cuda.synchronize()
    for k, v in (("y", y), ("dx", dx), ("dw", dw), ("db", db)):
        np.testing.assert_array_equal(v.cpu().numpy(), ref[k], err_msg=k)


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
@pytest.mark.parametrize("shape", [SHAPES[0], SHAPES[2], SHAPES[5], SHAPES[6]], ids=lambda s: s[0])
def test_single_cta_mma_path(shape, math):
    """Plan option cta_pairs = 0 forces single-CTA tcgen05 MMAs (no CTA pairs): still bit-exact on
    integer data, and equal to the default (paired) plan on random data (same per-element K order)."""
    d = _data(shape, exact=True, seed=21)
    got = _run(_layer(shape, math, cta_pairs=0), d)
    ref = _oracle(d, shape[7], shape[8])
    for k in ref:
        np.testing.assert_array_equal(got[k], ref[k].astype(np.float32), err_msg=k)
    dr = _data(shape, seed=22)
    one = _run(_layer(shape, math, cta_pairs=0), dr)
    two = _run(_layer(shape, math), dr)
    for k in ("y", "dx"):
        np.testing.assert_array_equal(one[k], two[k], err_msg=k)


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
@pytest.mark.parametrize("shape", [("c64_k3", 2, 64, 8, 8, 128, 3, 1, 1),
                                   ("c64_k3_n256", 2, 64, 8, 8, 256, 3, 1, 1),
                                   ("c96_k5", 2, 96, 9, 9, 256, 5, 1, 2),
                                   ("c256_k3_n384", 2, 256, 7, 7, 384, 3, 1, 1)],
                         ids=lambda s: s[0])
@pytest.mark.parametrize("cg2", ["0", "1"])
def test_wgrad_cta_pairs_exact(shape, math, cg2):
    """Filter gradient with and without CTA pairs (cta_group::2, MN-major halves of B; the
    C_o = 384 case switches to 64-byte rows so bn/2 = 96 is whole atoms) is bit-exact on integer
    data, with the split partials reduced at the paired row pitch."""
    d = _data(shape, exact=True, seed=41)
    got = _run(_layer(shape, math, wgrad_cta_pairs=int(cg2)), d)
    ref = _oracle(d, shape[7], shape[8])
    np.testing.assert_array_equal(got["dw"], ref["dw"].astype(np.float32))
    np.testing.assert_array_equal(got["db"], ref["db"].astype(np.float32))


# space-to-depth layers whose filter gradient runs on the shared-halo kernel (hwgrad.cuh)
HALO_SHAPES = [
    ("caffenet_conv1_full_hw", 2, 3, 227, 227, 96, 11, 4, 0),   # 9 taps (odd: duplicate pair)
    ("caffenet_conv1_s4", 2, 3, 67, 67, 96, 11, 4, 0),
    ("s2d_c12_k5_s2", 3, 12, 20, 21, 40, 5, 2, 2),             # 9 taps, C_o = 40 (one B atom)
    ("s2d_c16_k3_s2", 2, 16, 17, 15, 24, 3, 2, 1),             # 4 taps, no duplicate
    ("s2d_co112_k3_s2", 2, 16, 17, 15, 112, 3, 2, 1),          # C_o in (96, 128]: 2 dy builder groups
]


@pytest.mark.parametrize("shape", HALO_SHAPES, ids=lambda s: s[0])
def test_halo_wgrad_exact(shape):
    """The shared-halo filter gradient (row-shifted SWIZZLE_128B descriptors over one staged x'
    tile per k-block, dy on the padded grid) is bit-exact on integer data, and so is the
    backward-data pass that reads the padded dy; halo_wgrad = 0 (im2col path) agrees bit for bit."""
    d = _data(shape, exact=True, seed=43)
    ref = _oracle(d, shape[7], shape[8])
    layer = _layer(shape, "bf16")
    assert layer.info.wgrad_halo == 1
    got = _run(layer, d)
    for k in ("y", "dx", "dw", "db"):
        np.testing.assert_array_equal(got[k], ref[k].astype(np.float32), err_msg=k)
    layer0 = _layer(shape, "bf16", halo_wgrad=0)
    assert layer0.info.wgrad_halo == 0
    got0 = _run(layer0, d)
    for k in ("dw", "db", "dx"):
        np.testing.assert_array_equal(got0[k], got[k], err_msg=k)


@pytest.mark.parametrize("shape", HALO_SHAPES[:2], ids=lambda s: s[0])
def test_halo_wgrad_random_and_invariant(shape):
    """Random data: within the bf16 bar of the oracle and of the rounding-emulated oracle, and
    bitwise identical across samples-in-flight overrides and reruns (shape-only splits)."""
    d = _data(shape, seed=44)
    ref = _oracle(d, shape[7], shape[8])
    emu = _oracle(d, shape[7], shape[8], x=EMU["bf16"](d["x"]), w=EMU["bf16"](d["w"]),
                  dy=EMU["bf16"](d["dy"]))
    runs = [_run(_layer(shape, "bf16", S), d) for S in (0, 1, 2, 0)]
    for k in ("dw", "db"):
        r = ref[k]
        assert np.abs(runs[0][k] - r).max() / np.abs(r).max() <= TOL["bf16"], k
        e = emu[k]
        assert np.abs(runs[0][k] - e).max() / np.abs(e).max() <= 1e-4, k
        for other in runs[1:]:
            np.testing.assert_array_equal(other[k], runs[0][k], err_msg=k)


@pytest.mark.parametrize("shape", HALO_SHAPES, ids=lambda s: s[0])
def test_halo_wgrad_fused_dy(shape):
    """Fused-dy halo filter gradient (hwgrad_kernel<true>: the CTA's own warps build the dy
    operand from fp32 NCHW with the pack's RNE rounding, and emit the db partials): dW bitwise
    equal to the packed-dy kernel (fused_dy = 0: same operand bits, same MMA order), db within
    fp32 summation-order noise of it; the staged calls (GLP_PACK_DY_DB only records dy,
    bwd_data packs it lazily) bitwise equal to the composed calls."""
    d = _data(shape, seed=49)
    layer = _layer(shape, "bf16")
    assert layer.info.wgrad_fused_dy == 1
    ref = _run(layer, d)
    t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
    dx = torch.empty(layer.x_shape, device=DEV)
    dw = torch.empty(layer.w_shape, device=DEV)
    db = torch.empty(layer.geom.Co, device=DEV)
    layer.stage_pack(glp.GLP_PACK_X, t["x"])
    layer.stage_pack(glp.GLP_PACK_DY_DB, t["dy"])
    layer.stage_pack(glp.GLP_PACK_W_BWD_DATA, t["w"])
    layer.stage_bwd_filter()
    layer.stage_reduce(dw, db)
    layer.stage_bwd_data(dx)
    torch.cuda.synchronize()
    for k, v in (("dx", dx), ("dw", dw), ("db", db)):
        np.testing.assert_array_equal(v.cpu().numpy(), ref[k], err_msg=k)
    layer0 = _layer(shape, "bf16", fused_dy=0)
    assert layer0.info.wgrad_fused_dy == 0 and layer0.info.wgrad_halo == 1
    got0 = _run(layer0, d)
    np.testing.assert_array_equal(got0["dw"], ref["dw"])
    np.testing.assert_array_equal(got0["dx"], ref["dx"])
    scale = np.abs(d["dy"].astype(np.float64)).sum(axis=(0, 2, 3))
    assert np.all(np.abs(got0["db"].astype(np.float64) - ref["db"]) <= 1e-6 * scale)


@pytest.mark.parametrize("shape", HALO_SHAPES, ids=lambda s: s[0])
def test_halo_fwd_exact(shape):
    """The shared-halo forward (hfwd.cuh: one staged x' tile per 128 rows of the padded grid,
    row-shifted K-major SWIZZLE_128B descriptors per tap, resident W', invalid padded-grid rows
    dropped) is bit-exact on integer data, and halo_fwd = 0 (im2col forward) agrees bit for bit."""
    d = _data(shape, exact=True, seed=47)
    ref = _oracle(d, shape[7], shape[8])
    layer = _layer(shape, "bf16")
    assert layer.info.fwd_halo == 1
    got = _run(layer, d)
    np.testing.assert_array_equal(got["y"], ref["y"].astype(np.float32))
    layer0 = _layer(shape, "bf16", halo_fwd=0)
    assert layer0.info.fwd_halo == 0
    got0 = _run(layer0, d)
    np.testing.assert_array_equal(got0["y"], got["y"])


@pytest.mark.parametrize("shape", HALO_SHAPES[:3], ids=lambda s: s[0])
def test_halo_fwd_random_and_invariant(shape):
    """Random data: y within the bf16 bar of the oracle and 1e-4 of the rounding-emulated oracle,
    bitwise identical across samples-in-flight overrides (grid sizes) and reruns, and equal to
    the im2col forward (same MMA order: taps in order, 4 K=16 steps per 64-channel atom)."""
    d = _data(shape, seed=48)
    ref = _oracle(d, shape[7], shape[8])["y"]
    emu = _oracle(d, shape[7], shape[8], x=EMU["bf16"](d["x"]), w=EMU["bf16"](d["w"]),
                  dy=EMU["bf16"](d["dy"]))["y"]
    runs = [_run(_layer(shape, "bf16", S), d)["y"] for S in (0, 1, 2, 0)]
    assert np.abs(runs[0] - ref).max() / np.abs(ref).max() <= TOL["bf16"]
    assert np.abs(runs[0] - emu).max() / np.abs(emu).max() <= 1e-4
    for other in runs[1:]:
        np.testing.assert_array_equal(other, runs[0])
    np.testing.assert_array_equal(_run(_layer(shape, "bf16", halo_fwd=0), d)["y"], runs[0])


# fused sibling groups (include/glp.h): name, N, C, H, W, branches, K, S, P
GROUPS = [
    ("gnet_5b_1x1_siblings", 4, 832, 7, 7, [384, 192, 48], 1, 1, 0),
    ("k3_three_branches", 3, 64, 9, 11, [40, 24, 20], 3, 1, 1),
    ("k5_two_branches_ragged", 2, 32, 12, 12, [16, 50], 5, 1, 2),
]


def _group_data(g, exact, seed):
    _, N, C, H, W, br, K, S, P = g
    d = _data((None, N, C, H, W, sum(br), K, S, P), exact=exact, seed=seed)
    offs = np.cumsum([0] + br)
    split = lambda a, axis: [np.ascontiguousarray(np.take(a, range(offs[i], offs[i + 1]), axis=axis))
                             for i in range(len(br))]
    return d, split(d["w"], 0), split(d["b"], 0), split(d["dy"], 1)


def _group_run(layer, x, ws, bs, dys, staged=False):
    T = lambda a: torch.from_numpy(a).to(DEV)
    x_t, ws_t, bs_t, dys_t = T(x), [T(w) for w in ws], [T(b) for b in bs], [T(a) for a in dys]
    ys = [torch.full(s, float("nan"), device=DEV) for s in layer.branch_y_shapes()]
    dws = [torch.full(s, float("nan"), device=DEV) for s in layer.branch_w_shapes()]
    dbs = [torch.full((c,), float("nan"), device=DEV) for c in layer.branches]
    dx = torch.full(layer.x_shape, float("nan"), device=DEV)
    if staged:
        layer.stage_pack_group(glp.GLP_PACK_X, [x_t])
        layer.stage_pack_group(glp.GLP_PACK_W_FWD, ws_t)
        layer.stage_fwd_group(bs_t, ys)
        layer.stage_pack_group(glp.GLP_PACK_DY_DB, dys_t)
        layer.stage_pack_group(glp.GLP_PACK_W_BWD_DATA, ws_t)
        layer.stage_bwd_data(dx)
        layer.stage_bwd_filter()
        layer.stage_reduce_group(dws, dbs)
    else:
        layer.group_fwd(x_t, ws_t, bs_t, ys)
        layer.group_bwd(x_t, dys_t, ws_t, dx, dws, dbs)
    torch.cuda.synchronize()
    c = lambda l: [t.cpu().numpy() for t in l]
    return {"y": c(ys), "dx": dx.cpu().numpy(), "dw": c(dws), "db": c(dbs)}


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
@pytest.mark.parametrize("g", GROUPS, ids=lambda g: g[0])
def test_group_exact_vs_oracle(g, math):
    """A fused group equals the oracle of each branch bit for bit on integer data (y_b, dW_b,
    db_b per branch; dx = the sum of the branches' backward-data results)."""
    _, N, C, H, W, br, K, S, P = g
    d, ws, bs, dys = _group_data(g, True, 51)
    layer = glp.ConvLayer(N, C, H, W, None, K, S, P, math=math, branches=br)
    got = _group_run(layer, d["x"], ws, bs, dys)
    dx_ref = np.zeros(d["x"].shape)
    for i in range(len(br)):
        y = oracle.conv_fwd(d["x"], ws[i], bs[i], S, P)
        dw, _ = oracle.conv_bwd_filter(d["x"], dys[i], ws[i].shape, S, P)
        dx_ref += oracle.conv_bwd_data(dys[i], ws[i], d["x"].shape, S, P)
        np.testing.assert_array_equal(got["y"][i], y.astype(np.float32), err_msg=f"y{i}")
        np.testing.assert_array_equal(got["dw"][i], dw.astype(np.float32), err_msg=f"dw{i}")
        np.testing.assert_array_equal(got["db"][i], dys[i].astype(np.float64).sum(axis=(0, 2, 3)).astype(np.float32),
                                      err_msg=f"db{i}")
    np.testing.assert_array_equal(got["dx"], dx_ref.astype(np.float32))


@pytest.mark.parametrize("g", GROUPS, ids=lambda g: g[0])
def test_group_equals_concatenated_layer(g):
    """Random data: the per-branch group calls (composed and staged) are bitwise identical to the
    single-tensor calls of the same plan on the concatenated tensors, and within the bf16 bar of
    the oracle."""
    _, N, C, H, W, br, K, S, P = g
    d, ws, bs, dys = _group_data(g, False, 52)
    layer = glp.ConvLayer(N, C, H, W, None, K, S, P, math="bf16", branches=br)
    got = _group_run(layer, d["x"], ws, bs, dys)
    got_staged = _group_run(layer, d["x"], ws, bs, dys, staged=True)
    cat = _run(layer, d)
    offs = np.cumsum([0] + br)
    for i in range(len(br)):
        for k, axis in (("y", 1), ("dw", 0), ("db", 0)):
            ref = np.take(cat[k], range(offs[i], offs[i + 1]), axis=axis)
            np.testing.assert_array_equal(got[k][i], ref, err_msg=f"{k}{i}")
            np.testing.assert_array_equal(got_staged[k][i], ref, err_msg=f"staged {k}{i}")
    np.testing.assert_array_equal(got["dx"], cat["dx"])
    np.testing.assert_array_equal(got_staged["dx"], cat["dx"])
    ref = _oracle(d, S, P)
    for k in ("y", "dx", "dw", "db"):
        assert np.abs(cat[k] - ref[k]).max() / np.abs(ref[k]).max() <= TOL["bf16"], k


def test_group_rejects_misaligned_branch():
    """Every branch but the last must start on a 16-byte chunk of the packed pitch."""
    with pytest.raises(glp.GlpError):
        glp.ConvLayer(2, 16, 8, 8, None, 3, 1, 1, math="bf16", branches=[12, 20])
    glp.ConvLayer(2, 16, 8, 8, None, 3, 1, 1, math="bf16", branches=[16, 20])   # ok


POOL_SHAPES = [SHAPES[0], SHAPES[2], SHAPES[6], ("k5_ragged", 5, 24, 11, 13, 40, 5, 1, 2)]


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32", "fp32_simt"])
@pytest.mark.parametrize("shape", POOL_SHAPES, ids=lambda s: s[0])
def test_stream_pool_comparator(shape, math):
    """The paper's per-sample stream pool (prior-art comparator): forward and backward-data are
    bitwise the batched persistent path's results; the filter gradient is bit-exact on integer
    data and within the tolerance on random data; the pool size is the Eq. 7 bound unless set."""
    _, N, C, H, W, Co, K, S, P = shape
    T = lambda a: torch.from_numpy(a).to(DEV)
    for exact, seed in ((True, 61), (False, 62)):
        d = _data(shape, exact=exact, seed=seed)
        ref_layer = _run(_layer(shape, math), d)
        for ns in (0, 3):
            pool = glp.StreamPool(N, C, H, W, Co, K, S, P, math=math, n_streams=ns)
            assert pool.n_streams == (min(pool.eq7_bound, N) if ns == 0 else min(3, N))
            y = torch.full(ref_layer["y"].shape, float("nan"), device=DEV)
            dx = torch.full(ref_layer["dx"].shape, float("nan"), device=DEV)
            dw = torch.full(ref_layer["dw"].shape, float("nan"), device=DEV)
            db = torch.full(ref_layer["db"].shape, float("nan"), device=DEV)
            pool.fwd(T(d["x"]), T(d["w"]), T(d["b"]), y)
            pool.bwd(T(d["x"]), T(d["dy"]), T(d["w"]), dx, dw, db)
            torch.cuda.synchronize()
            got = {"y": y.cpu().numpy(), "dx": dx.cpu().numpy(), "dw": dw.cpu().numpy(),
                   "db": db.cpu().numpy()}
            np.testing.assert_array_equal(got["y"], ref_layer["y"])
            np.testing.assert_array_equal(got["dx"], ref_layer["dx"])
            if exact:
                ref = _oracle(d, S, P)
                for k in ("dw", "db"):
                    np.testing.assert_array_equal(got[k], ref[k].astype(np.float32), err_msg=k)
            else:
                for k in ("dw", "db"):
                    r = ref_layer[k]
                    assert np.abs(got[k] - r).max() / np.abs(r).max() <= TOL[math], k


# Caffe convolution groups (glp_conv_desc_set_groups): name, N, C, H, W, Co,
# K, S, P, groups
GROUPED = [
    ("caffenet_conv2_g2", 2, 96, 27, 27, 256, 5, 1, 2, 2),
    ("caffenet_conv4_g2", 3, 384, 13, 13, 384, 3, 1, 1, 2),
    ("s4_k11_g3", 2, 6, 35, 35, 48, 11, 4, 0, 3),     # space-to-depth + halo per group
    ("g4_ragged", 3, 32, 9, 11, 40, 3, 2, 1, 4),
]


def _grouped_oracle(d, S, P, G):
    x, w, b, dy = d["x"], d["w"], d["b"], d["dy"]
    C, Co = x.shape[1], w.shape[0]
    cg, og = C // G, Co // G
    out = {"y": [], "dx": [], "dw": [], "db": []}
    for g in range(G):
        xs, ws_ = x[:, g * cg:(g + 1) * cg], w[g * og:(g + 1) * og]
        dys = dy[:, g * og:(g + 1) * og]
        out["y"].append(oracle.conv_fwd(xs, ws_, b[g * og:(g + 1) * og], S, P))
        out["dx"].append(oracle.conv_bwd_data(dys, ws_, xs.shape, S, P))
        out["dw"].append(oracle.conv_bwd_filter(xs, dys, ws_.shape, S, P)[0])
    return {"y": np.concatenate(out["y"], 1), "dx": np.concatenate(out["dx"], 1),
            "dw": np.concatenate(out["dw"], 0), "db": dy.astype(np.float64).sum(axis=(0, 2, 3))}


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32", "fp32_simt"])
@pytest.mark.parametrize("shape", GROUPED, ids=lambda s: s[0])
def test_grouped_conv(shape, math):
    """Grouped convolution equals the oracle of each group: bit-exact on integer data (every
    math mode), within the bar on random data; the staged calls equal the composed ones."""
    _, N, C, H, W, Co, K, S, P, G = shape
    Ho, Wo = oracle.out_dim(H, K, S, P), oracle.out_dim(W, K, S, P)
    for exact, seed in ((True, 71), (False, 72)):
        d = gen_custom(N, C // G, H, W, Co, K, K, seed, exact=exact, Ho=Ho, Wo=Wo)
        d["x"] = gen_custom(N, C, H, W, Co, K, K, seed + 100, exact=exact, Ho=Ho, Wo=Wo)["x"]
        layer = glp.ConvLayer(N, C, H, W, Co, K, S, P, math=math, groups=G)
        assert layer.w_shape == d["w"].shape
        got = _run(layer, d)
        ref = _grouped_oracle(d, S, P, G)
        for k in ("y", "dx", "dw", "db"):
            if exact:
                np.testing.assert_array_equal(got[k], ref[k].astype(np.float32), err_msg=k)
            else:
                assert np.abs(got[k] - ref[k]).max() / np.abs(ref[k]).max() <= TOL[math], k
    if math != "fp32_simt":
        t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
        y = torch.empty(layer.y_shape, device=DEV)
        dx = torch.empty(layer.x_shape, device=DEV)
        dw = torch.empty(layer.w_shape, device=DEV)
        db = torch.empty(Co, device=DEV)
        layer.stage_pack(glp.GLP_PACK_X, t["x"])
        layer.stage_pack(glp.GLP_PACK_W_FWD, t["w"])
        layer.stage_fwd(t["b"], y)
        layer.stage_pack(glp.GLP_PACK_DY_DB, t["dy"])
        layer.stage_pack(glp.GLP_PACK_W_BWD_DATA, t["w"])
        layer.stage_bwd_data(dx)
        layer.stage_bwd_filter()
        layer.stage_reduce(dw, db)
        torch.cuda.synchronize()
        for k, v in (("y", y), ("dx", dx), ("dw", dw), ("db", db)):
            np.testing.assert_array_equal(v.cpu().numpy(), got[k], err_msg="staged " + k)


@pytest.mark.parametrize("shape", [(16, 24, 8, 8, 40, 3, 1, 1), (16, 1, 36, 36, 20, 5, 1, 0)],
                         ids=["c24k3", "small_filter"])
@pytest.mark.parametrize("math", ["fp32", "tf32", "bf16"])
def test_tree_exchange_bitwise_invariant_emulated_ranks(math, shape):
    """Deterministic gradient exchange (NEXT-2) as the library runs it, with 1, 2, 4 and 8 ranks
    emulated on one device: each rank plans its local batch as 8/world leaves (wgrad_leaves),
    packs x and dy ONCE, runs one filter-gradient GEMM whose splits never cross a leaf, reduces
    per leaf (glp_stage_reduce_leaves), sums its leaves with glp_tree_sum (its subtree of the
    8-leaf tree), and glp_tree_exchange -- called once per emulated rank with every rank's
    buffers as the "peer" pointers -- completes the top of the tree into every rank's output.
    dW||db is bitwise the same for every world size and every rank, equal to the composed
    glp_conv_bwd_filter of the 8-leaf plan, within the bar of the oracle, exact on integers.
    small_filter (C*K*K = 25, leaf = 2 images x 1024 pixels): the per-leaf dW reductions run the
    8-phase small-filter kernel (grid z = leaf)."""
    from paper_conf_icpp_futhys18_b200.dist import LEAVES, rank_leaves
    N, C, H, W, Co, K, S, P = shape
    Ho = oracle.out_dim(H, K, S, P)
    wsz = Co * C * K * K
    numel = (wsz + Co + 3) // 4 * 4
    for exact, seed in ((False, 81), (True, 82)):
        d = gen_custom(N, C, H, W, Co, K, K, seed, exact=exact, Ho=Ho, Wo=Ho)
        t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
        results = []
        for world in (1, 2, 4, 8):
            nl = N // world
            subs, outs = [], []
            for r in range(world):
                L = len(rank_leaves(r, world))
                layer = glp.ConvLayer(nl, C, H, W, Co, K, S, P, math=math,
                                      options={"wgrad_leaves": L})
                leaves = torch.zeros(L, numel, device=DEV)
                flat = leaves.view(-1)
                layer.stage_pack(glp.GLP_PACK_X, t["x"][r * nl:(r + 1) * nl].contiguous())
                layer.stage_pack(glp.GLP_PACK_DY_DB, t["dy"][r * nl:(r + 1) * nl].contiguous())
                layer.stage_bwd_filter()
                layer.stage_reduce_leaves(flat, flat[wsz:], numel)
                sub = torch.empty(numel, device=DEV)
                glp.tree_sum([leaves[l] for l in range(L)], sub)
                subs.append(sub)
                outs.append(torch.full((numel,), float("nan"), device=DEV))
            for r in range(world):
                glp.tree_exchange([x.data_ptr() for x in subs], [o.data_ptr() for o in outs], r, numel)
            torch.cuda.synchronize()
            for o in outs[1:]:
                np.testing.assert_array_equal(o.cpu().numpy(), outs[0].cpu().numpy())
            results.append(outs[0].cpu().numpy())
        for r in results[1:]:
            np.testing.assert_array_equal(r, results[0])
        # the composed call of the 8-leaf plan (leaves reduced in the workspace, the same tree)
        layer = glp.ConvLayer(N, C, H, W, Co, K, S, P, math=math, options={"wgrad_leaves": LEAVES})
        if C == 1 and math != "bf16":
            assert layer.info.wgrad_reduce_wide == 1
        dw = torch.empty(layer.w_shape, device=DEV)
        db = torch.empty(Co, device=DEV)
        layer.bwd_filter(t["x"], t["dy"], dw, db)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(dw.cpu().numpy().ravel(), results[0][:wsz])
        np.testing.assert_array_equal(db.cpu().numpy(), results[0][wsz:wsz + Co])
        rdw, rdb = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, S, P)
        full = np.concatenate([rdw.ravel(), rdb])
        if exact:
            np.testing.assert_array_equal(results[0][:wsz + Co], full.astype(np.float32))
        else:
            assert oracle.normwise_err(results[0][:wsz + Co], full) <= TOL[math]


def test_tree_sum_matches_sum2_tree():
    """glp_tree_sum (one launch) is bitwise the dist.tree_sum of glp_sum2 adds, for 1-8 parts."""
    from paper_conf_icpp_futhys18_b200.dist import tree_sum
    g = torch.Generator(device="cpu").manual_seed(5)
    for n in (1, 2, 4, 8):
        parts = [(torch.randn(5003, generator=g) * 10.0 ** torch.empty(5003).uniform_(-6, 6,
                  generator=g)).to(DEV) for _ in range(n)]
        ref = tree_sum(parts, lambda a, b, o: glp.sum2(a, b, o))
        out = torch.empty_like(parts[0])
        glp.tree_sum(parts, out)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(out.cpu().numpy(), ref.cpu().numpy())


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
@pytest.mark.parametrize("shape", [SHAPES[0], SHAPES[4], SHAPES[5], SHAPES[6], SHAPES[1], SHAPES[9]],
                         ids=lambda s: s[0])
def test_pack_w_both_equals_separate(shape, math):
    """GLP_PACK_W_BOTH (both weight operands from one pass over W) writes the same operand bits
    as GLP_PACK_W_FWD + GLP_PACK_W_BWD_DATA: the staged forward and backward-data outputs are
    bitwise equal (channel padding C, C_o % 32 != 0, 1x1 / 3x3 / 5x5 taps)."""
    d = _data(shape, seed=51)
    t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
    outs = []
    for both in (False, True):
        layer = _layer(shape, math)
        y = torch.empty(layer.y_shape, device=DEV)
        dx = torch.empty(layer.x_shape, device=DEV)
        layer.stage_pack(glp.GLP_PACK_X, t["x"])
        if both:
            layer.stage_pack(glp.GLP_PACK_W_BOTH, t["w"])
        else:
            layer.stage_pack(glp.GLP_PACK_W_FWD, t["w"])
            layer.stage_pack(glp.GLP_PACK_W_BWD_DATA, t["w"])
        layer.stage_fwd(t["b"], y)
        layer.stage_pack(glp.GLP_PACK_DY, t["dy"])
        layer.stage_bwd_data(dx)
        torch.cuda.synchronize()
        outs.append((y.cpu().numpy(), dx.cpu().numpy()))
    np.testing.assert_array_equal(outs[1][0], outs[0][0])
    np.testing.assert_array_equal(outs[1][1], outs[0][1])


# unit-stride layers for the shared-halo backward-data kernel (hdgrad.cuh); halo_dgrad = 2 forces it
# where the cost model would keep the im2col kernel (small images waste more padded rows)
HDG_SHAPES = [
    ("caffenet_conv2_b2", 2, 96, 27, 27, 256, 5, 1, 2),     # the model's own choice; odd unit count
    ("k3p1_ragged", 3, 64, 11, 13, 64, 3, 1, 1),            # 3 images x 2 tiles: ragged pair unit
    ("k3p0", 2, 32, 10, 12, 64, 3, 1, 0),                   # dy smaller than dx: halo offset Q = 2
    ("k5p1", 2, 32, 9, 9, 128, 5, 1, 1),                    # asymmetric halo (Q = 3)
]


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
@pytest.mark.parametrize("shape", HDG_SHAPES, ids=lambda s: s[0])
def test_halo_dgrad(shape, math):
    """Shared-halo backward-data (4-D TMA halo of the packed dy per 128-byte channel block -- 64
    bf16 / 32 tf32 channels -- flipped taps by row shift, CTA pairs with M = 256 MMAs): bit-exact
    on integer data, within 1e-4 of the rounding-emulated oracle and the mode's bar of the fp64
    oracle on random data, bitwise invariant across samples-in-flight overrides.  fp32: the mixed
    split (fp32_split = 1: tf32 hi and two bf16 halo tiles per channel block, the 64-byte bf16
    rows shifted like the tf32 ones, chunked accumulation) against 1e-5 of the fp64 oracle and
    5e-6 of the oracle of the split's own products."""
    opts = dict(halo_dgrad=2, **({"fp32_split": 1} if math == "fp32" else {}))
    layer = _layer(shape, math, **opts)
    assert layer.info.dgrad_halo == 1
    if math == "fp32":
        assert layer.info.fp32_split == 1
    d = _data(shape, exact=True, seed=53)
    got = _run(layer, d)
    ref = _oracle(d, shape[7], shape[8])
    np.testing.assert_array_equal(got["dx"], ref["dx"].astype(np.float32))
    d = _data(shape, seed=54)
    runs = [_run(_layer(shape, math, S, **opts), d)["dx"] for S in (0, 1, 0)]
    ref = _oracle(d, shape[7], shape[8])["dx"]
    if math == "fp32":
        emu, bar = _mixed_emulated(d, shape[7], shape[8])["dx"], 5e-6
    else:
        emu = _oracle(d, shape[7], shape[8], x=EMU[math](d["x"]), w=EMU[math](d["w"]),
                      dy=EMU[math](d["dy"]))["dx"]
        bar = 1e-4
    assert np.abs(runs[0] - ref).max() / np.abs(ref).max() <= TOL[math]
    assert np.abs(runs[0] - emu).max() / np.abs(emu).max() <= bar
    for other in runs[1:]:
        np.testing.assert_array_equal(other, runs[0])


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
def test_strided_dgrad_space_to_depth(math):
    """Strided layers whose forward runs on the space-to-depth x' (CaffeNet conv1, ragged_s2) take
    the backward-data as the stride-1 backward-data of that form (dx' over x', then scattered into
    dx; dgrad_s2d = 1): bit-exact on integer data against the oracle's col2im, which is written
    for the strided layer itself (the exactness and emulated-rounding cases of SHAPES cover the
    random data)."""
    for shape in (SHAPES[2], SHAPES[3]):
        layer = _layer(shape, math)
        assert layer.info.dgrad_s2d == 1, shape[0]
        d = _data(shape, exact=True, seed=57)
        got = _run(layer, d)
        ref = _oracle(d, shape[7], shape[8])
        np.testing.assert_array_equal(got["dx"], ref["dx"].astype(np.float32), err_msg=shape[0])
    # the staged calls (the bench's path; bf16 conv1 packs dy lazily for its fused-dy filter
    # gradient) give the same dx bits
    shape = SHAPES[2]
    layer = _layer(shape, math)
    d = _data(shape, exact=True, seed=57)
    t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
    dx = torch.full(layer.x_shape, float("nan"), device=DEV)
    layer.stage_pack(glp.GLP_PACK_W_BWD_DATA, t["w"])
    layer.stage_pack(glp.GLP_PACK_DY, t["dy"])
    layer.stage_bwd_data(dx)
    torch.cuda.synchronize()
    ref = _oracle(d, shape[7], shape[8])
    np.testing.assert_array_equal(dx.cpu().numpy(), ref["dx"].astype(np.float32))
    # unit-stride layers keep their own backward-data
    assert _layer(SHAPES[6], math).info.dgrad_s2d == 0


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
def test_pack_variants_same_operands(math):
    """The warp-tiled and the block-tiled activation packs (plan option pack_block; the default
    takes the block-tiled one for 4-byte operands) write the same operand bits: y, dx and dW are
    bitwise equal; db (summed per row tile of the pack, 32 vs 128 rows) within summation-order
    noise."""
    for shape in (SHAPES[0], MIX_SHAPES[2], SHAPES[2]):
        d = _data(shape, seed=58)
        a = _run(_layer(shape, math, pack_block=0), d)
        b = _run(_layer(shape, math, pack_block=1), d)
        for k in ("y", "dx", "dw"):
            np.testing.assert_array_equal(a[k], b[k], err_msg=f"{shape[0]} {k}")
        scale = np.abs(d["dy"].astype(np.float64)).sum(axis=(0, 2, 3))
        assert np.all(np.abs(a["db"].astype(np.float64) - b["db"]) <= 1e-6 * scale), shape[0]


def test_halo_dgrad_model_choice():
    """The cost model picks the halo backward-data for CaffeNet conv2 (27x27, 5x5, C_i = 96) in bf16
    and tf32, keeps the im2col kernel for the 13x13 layers (conv3-5: half of the padded rows would
    be junk), for 3xTF32 (no two-plane halo kernel) and for the mixed fp32 split (its halo kernel
    measured slower than the im2col one on conv2: opt-in with halo_dgrad = 2)."""
    for math in ("bf16", "tf32"):
        assert _layer(HDG_SHAPES[0], math).info.dgrad_halo == 1
        assert _layer(SHAPES[6], math).info.dgrad_halo == 0
    assert _layer(HDG_SHAPES[0], "fp32", fp32_split=1).info.dgrad_halo == 0
    assert _layer(HDG_SHAPES[0], "fp32", fp32_split=1, halo_dgrad=2).info.dgrad_halo == 1
    assert _layer(HDG_SHAPES[0], "fp32", fp32_split=0).info.dgrad_halo == 0


@pytest.mark.parametrize("ncg", ["1", "2"])
def test_halo_wgrad_fused_dy_variants(ncg):
    """The other fused-dy builder variants (fused_dy_builders = 1: cp.async landing zone; 2: two
    register groups) give the same dW bits as the default and db within summation-order noise."""
    shape = HALO_SHAPES[1]
    d = _data(shape, seed=55)
    ref = _run(_layer(shape, "bf16"), d)
    layer = _layer(shape, "bf16", fused_dy_builders=int(ncg))
    assert layer.info.wgrad_fused_dy == 1
    got = _run(layer, d)
    np.testing.assert_array_equal(got["dw"], ref["dw"])
    scale = np.abs(d["dy"].astype(np.float64)).sum(axis=(0, 2, 3))
    assert np.all(np.abs(got["db"].astype(np.float64) - ref["db"]) <= 1e-6 * scale)


LONG_K = [("caffenet_conv2", 2, 96, 27, 27, 256, 5, 1, 2),    # dgrad K = 6400, fwd K = 2400
          ("caffenet_conv4", 2, 384, 13, 13, 384, 3, 1, 1),   # K = 3456 both ways
          ("gnet_conv_4", 3, 192, 7, 7, 384, 3, 1, 1)]


@pytest.mark.parametrize("split", [0, 1], ids=["3xtf32", "mixed"])
@pytest.mark.parametrize("shape", LONG_K, ids=lambda s: s[0])
def test_fp32_long_reductions(shape, split):
    """GLP_MATH_FP32 (3xTF32, and the mixed split) at the paper's longest reductions: the tensor
    core truncates each MMA's fp32 result, so the error of one TMEM accumulator grows with K; the
    chunked fp32 register accumulation keeps every output within the 1e-5 normwise bar
    (BASELINE.json north_star)."""
    d = _data(shape, seed=91)
    layer = _layer(shape, "fp32", fp32_split=split)
    assert layer.info.fp32_split == split
    got = _run(layer, d)
    ref = _oracle(d, shape[7], shape[8])
    errs = {k: oracle.normwise_err(got[k], ref[k]) for k in ref}
    assert all(e <= TOL["fp32"] for e in errs.values()), errs


def test_binding_rejects_bad_tensors():
    """The Python binding checks every tensor before the C call (dtype, device, contiguity and the
    exact shape the kernels index): a wrong tensor raises ValueError instead of letting the
    kernels read or write past an allocation."""
    shape = SHAPES[0]
    layer = _layer(shape, "bf16")
    x = torch.zeros(layer.x_shape, device=DEV)
    w = torch.zeros(layer.w_shape, device=DEV)
    b = torch.zeros(layer.geom.Co, device=DEV)
    y = torch.zeros(layer.y_shape, device=DEV)
    bad = [
        (x.half(), w, b, y),                                   # dtype
        (x.cpu(), w, b, y),                                    # device
        (x.transpose(2, 3), w, b, y),                          # not contiguous
        (x, w, b, torch.zeros(layer.y_shape[0], layer.y_shape[1] + 1, *layer.y_shape[2:],
                              device=DEV)),                    # shape
        (x, w[:, :1].contiguous(), b, y),                      # weight shape
        (x, w, torch.zeros(layer.geom.Co + 1, device=DEV), y),  # bias shape
    ]
    for args in bad:
        with pytest.raises(ValueError):
            layer.fwd(*args)
    layer.fwd(x, w, None, y)   # bias is nullable
    with pytest.raises(ValueError):
        layer.bwd_filter(x, y, torch.zeros(1, device=DEV))


TABLE5 = [  # every Table 5 layer (P334-355) at its BASELINE.json batch
    ("lenet_conv1", 64, 1, 28, 28, 20, 5, 1, 0), ("lenet_conv2", 64, 20, 12, 12, 50, 5, 1, 0),
    ("cifar10_conv1", 100, 3, 32, 32, 32, 5, 1, 2), ("cifar10_conv2", 100, 32, 16, 16, 32, 5, 1, 2),
    ("cifar10_conv3", 100, 32, 8, 8, 64, 5, 1, 2),
    ("caffenet_conv1", 256, 3, 227, 227, 96, 11, 4, 0), ("caffenet_conv2", 256, 96, 27, 27, 256, 5, 1, 2),
    ("caffenet_conv3", 256, 256, 13, 13, 384, 3, 1, 1), ("caffenet_conv4", 256, 384, 13, 13, 384, 3, 1, 1),
    ("caffenet_conv5", 256, 384, 13, 13, 256, 3, 1, 1),
    ("googlenet_conv_1", 128, 160, 7, 7, 320, 3, 1, 1), ("googlenet_conv_2", 128, 832, 7, 7, 32, 1, 1, 0),
    ("googlenet_conv_3", 128, 832, 7, 7, 384, 1, 1, 0), ("googlenet_conv_4", 128, 192, 7, 7, 384, 3, 1, 1),
    ("googlenet_conv_5", 128, 832, 7, 7, 192, 1, 1, 0), ("googlenet_conv_6", 128, 832, 7, 7, 48, 1, 1, 0),
]


@pytest.mark.parametrize("math", ["bf16", "tf32", "fp32"])
def test_samples_in_flight_through_analyzer(math):
    """S (the paper's C_out, Eq. 9 re-derived, P254) of every Table 5 layer's plan equals the
    oracle analyzer's enumeration on the attributes of the forward kernel the plan launches:
    CTAs/SM by enumeration over every per-SM limit (TMEM charged whole, R16), resident rows =
    148 x CTAs/SM x 128, rows per sample = H_o*W_o x N tiles (the padded x' grid for the halo
    forward), S = largest s <= N with s * rows_per_sample <= resident rows (>= 1)."""
    from oracle import analyzer as A
    dev = A.B200()
    for shape in TABLE5:
        name, N, C, H, W, Co, K, St, P = shape
        layer = _layer(shape, math)
        info = layer.info
        a = layer.kernel_attr(0)
        beta = A.ctas_per_sm_enum(a["threads"], a["regs"], a["smem"], 512 if a["tmem_cols"] else 0, dev)
        slot_rows = dev.n_sm * beta * 128
        Ho = oracle.out_dim(H, K, St, P)
        if info.fwd_halo:
            Ks = -(-K // St)
            rows = (Ho + Ks - 1) * (Ho + Ks - 1)
        else:
            rows = Ho * Ho * -(-Co // info.tile_n_fwd)
        assert (info.s_slot_rows, info.s_rows_per_sample) == (slot_rows, rows), name
        assert info.samples_in_flight == A.samples_in_flight_enum(slot_rows, rows, N), name


def test_resource_tracker_records_plan_kernels():
    """The CUPTI resource tracker (NEXT-4; P165) records the kernels a call launches with the
    analyzer's inputs: the forward GEMM's grid, block, cluster, registers and shared memory equal
    the plan's, and launch-API durations (T_launch) are collected."""
    from paper_conf_icpp_futhys18_b200.tracker import Tracker
    shape = SHAPES[6]
    layer = _layer(shape, "bf16")
    d = _data(shape, seed=2)
    t = {k: torch.from_numpy(v).to(DEV) for k, v in d.items()}
    y = torch.empty(layer.y_shape, device=DEV)
    layer.fwd(t["x"], t["w"], t["b"], y)
    torch.cuda.synchronize()
    with Tracker() as tr:
        layer.fwd(t["x"], t["w"], t["b"], y)
    gemm = [k for k in tr.kernels if "igemm_kernel" in k.name]
    assert len(gemm) == 1, [k.name for k in tr.kernels]
    k, a = gemm[0], layer.kernel_attr(0)
    assert (k.grid[0], k.block[0], k.regs) == (layer.info.grid_fwd, a["threads"], a["regs"])
    assert k.cluster[0] in (1, 2) and k.smem >= a["smem"] and k.duration_us > 0
    assert any("pack" in r.name for r in tr.kernels)
    assert len(tr.launch_us) >= 3 and all(v > 0 for v in tr.launch_us)


@pytest.mark.parametrize("math", ["bf16", "fp32"])
def test_pool_eq7_launch_term(math):
    """The stream-pool comparator profiled once by the resource tracker: T_K (its per-sample
    forward GEMMs) and T_launch (launch API calls) give the Eq. 7 bound with the launch term
    (P245) exactly as the oracle's model computes it, the pool resizes to it, and its outputs
    keep the persistent path's bits."""
    from oracle import analyzer as A
    shape = SHAPES[0]
    _, N, C, H, W, Co, K, S, P = shape
    d = _data(shape, seed=3)
    T = lambda a: torch.from_numpy(a).to(DEV)
    pool = glp.StreamPool(N, C, H, W, Co, K, S, P, math=math)
    y = torch.empty((N, Co, oracle.out_dim(H, K, S, P), oracle.out_dim(W, K, S, P)), device=DEV)
    pool.fwd(T(d["x"]), T(d["w"]), T(d["b"]), y)
    tk, tl, recs = pool.calibrate(T(d["x"]), T(d["w"]), T(d["b"]), y)
    assert tk > 0 and tl > 0 and len(recs) == N   # one per-sample forward GEMM per sample
    one = glp.ConvLayer(1, C, H, W, Co, K, S, P, math=math)
    a = one.kernel_attr(0)
    kern = A.Kernel(blocks=one.info.grid_fwd, threads=a["threads"], smem=a["smem"],
                    t_kernel=tk, t_launch=tl)
    exp = max(1, min(A.eq7_bound(kern, A.B200()), A.B200().C))
    assert pool.eq7_launch_bound == exp
    assert pool.n_streams == max(1, min(exp, N, 64))
    y2 = torch.empty_like(y)
    pool.fwd(T(d["x"]), T(d["w"]), T(d["b"]), y2)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(y2.cpu().numpy(), _run(_layer(shape, math), d)["y"])
