"""Full-size parity: every BASELINE.json config at its full batch, run by bench.py itself (same
plans, same CUDA-graph-replayed step DAG it times; `--dump` saves each unit's inputs and outputs
after the timed steps), checked against the oracle on sampled outputs it computes one by one
(oracle.conv_fwd_at / conv_bwd_data_at / conv_bwd_filter_at) and on db in full.

Bars: integer data (`--exact-data`) -> every sampled element bit-exact; float
data -> |g - r| <= bar * max_sampled |r| against the fp64 oracle on the unrounded inputs (the
north_star bar, normwise over the sample: 2e-2 for TF32/BF16, 1e-5 for GLP_MATH_FP32 = 3xTF32)
and |g - r_emu| <= 1e-5 * sum|a||b| against the oracle of the products the MMAs form (operands
rounded as the pack step defines; 3xTF32: hi*hi + hi*lo + lo*hi of oracle.split_3xtf32) -- the
condition-aware bound of fp32 accumulation over exactly formed products.  Samples always include
the first and the last element (the ragged last tile) of every tensor.  db is compared in full
with oracle.conv_db.

test_fullsize_whole_tensor_exact: CaffeNet conv1-5 at batch 256 (BASELINE.json configs[3]) with
integer data, every output tensor compared WHOLE and bit for bit with the oracle, in every tensor
math mode (one oracle pass serves the three modes: the integer draws are the same).
"""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
EMU = {"tf32": oracle.round_tf32_rna, "bf16": oracle.round_bf16_rne}
BAR = {"bf16": 2e-2, "tf32": 2e-2, "fp32": 1e-5}
NS = 40   # sampled elements per tensor


def _bench_dump(tmp, workload, math, exact):
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--workload", str(workload), "--math",
           math, "--steps", "2", "--warmup", "3", "--no-cpu-baseline", "--no-e2e", "--dump", str(tmp)]
    if exact:
        cmd.append("--exact-data")
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["launch"].startswith("cuda_graph")
    return json.load(open(os.path.join(tmp, "meta.json")))


def _load(tmp, i, name):
    return np.load(os.path.join(tmp, f"u{i}_{name}.npy"), mmap_mode="r")


def _samples(shape, rng):
    idx = [tuple(0 for _ in shape), tuple(s - 1 for s in shape)]
    idx += [tuple(int(rng.integers(0, s)) for s in shape) for _ in range(NS - 2)]
    return idx


def _emu(fn, a, b, math, *rest, **kw):
    """Oracle value of the products the MMAs form from operands a, b (one element): the rounded
    operands (TF32 / BF16), or for 3xTF32 hi*hi + hi*lo + lo*hi of the split planes (the oracle
    is linear in each operand).  `a`, `b` are (array, rounded) pairs prepared by _prep."""
    if math != "fp32":
        return fn(a[1], b[1], *rest, **kw)
    (ah, al), (bh, bl) = a[2], b[2]
    return fn(ah, bh, *rest, **kw) + fn(ah, bl, *rest, **kw) + fn(al, bh, *rest, **kw)


def _prep(v, math):
    """(fp32 array, rounded operand, (hi, lo) split) of one operand."""
    if math == "fp32":
        hi, lo = oracle.split_3xtf32(v)
        return (v, hi, (hi, lo))
    return (v, EMU[math](v), None)


def _sl(p, *idx):
    """Slice every member of a _prep triple."""
    return (p[0][idx], p[1][idx], None if p[2] is None else (p[2][0][idx], p[2][1][idx]))


def _check(kind, got, ref, emu, scale, exact, math, what):
    got, ref = np.asarray(got, np.float64), np.asarray(ref, np.float64)
    if exact:
        np.testing.assert_array_equal(got, ref, err_msg=what)
        return
    bar = BAR[math] * max(np.abs(ref).max(), 1e-30)
    assert np.abs(got - ref).max() <= bar, (what, np.abs(got - ref).max() / bar * BAR[math])
    emu, scale = np.asarray(emu, np.float64), np.asarray(scale, np.float64)
    assert np.all(np.abs(got - emu) <= 1e-5 * scale + 1e-30), (
        what, float((np.abs(got - emu) / np.maximum(scale, 1e-30)).max()))


def _check_unit(tmp, i, u, math, exact, rng, extra=()):
    """extra: (x, dy) of the units that share this unit's parameters (Siamese towers): their
    filter gradients accumulate into this unit's dW / db (Caffe beta = 1)."""
    S, P, G = u["S"], u["P"], u["groups"]
    x = np.asarray(_load(tmp, i, "x"))
    grp = u["kind"] == "group"
    nb = len(u["Co"])
    xp = _prep(x, math)
    dx_terms = []
    for b in range(nb):
        sfx = str(b) if grp else ""
        w = np.asarray(_load(tmp, i, "w" + sfx))
        bias = np.asarray(_load(tmp, i, "b" + sfx))
        dy = np.asarray(_load(tmp, i, "dy" + sfx))
        y = _load(tmp, i, "y" + sfx)
        dw = _load(tmp, i, "dw" + sfx)
        db = _load(tmp, i, "db" + sfx)
        wp, dyp = _prep(w, math), _prep(dy, math)
        Cg, Cog = u["C"] // G, u["Co"][b] // G
        name = f"{u['names'][b]}"

        def grp_of(co):   # Caffe groups: output channel co reads input channels of its group
            g = co // Cog
            return g, slice(g * Cg, (g + 1) * Cg), slice(g * Cog, (g + 1) * Cog)

        # forward
        idx = _samples(y.shape, rng)
        g_, ref, emu, sc = [], [], [], []
        for n, co, ho, wo in idx:
            g, cs, _ = grp_of(co)
            xi = x[n:n + 1, cs]
            j = (0, co - g * Cog, ho, wo)
            wg = w[g * Cog:(g + 1) * Cog]
            bg = bias[g * Cog:(g + 1) * Cog]
            g_.append(y[n, co, ho, wo])
            ref.append(oracle.conv_fwd_at(xi, wg, bg, S, P, j))
            emu.append(_emu(oracle.conv_fwd_at, _sl(xp, slice(n, n + 1), cs),
                            _sl(wp, slice(g * Cog, (g + 1) * Cog)), math, None, S, P, j) + float(bg[j[1]]))
            sc.append(oracle.conv_fwd_at(xi, wg, None, S, P, j, absmode=True) + abs(float(bg[j[1]])))
        _check("y", g_, ref, emu, sc, exact, math, f"{name} y")
        if u.get("shares"):   # dW / db are the owner's (checked there, with this unit's share)
            dx_terms.append((w, wp, dy, dyp, Cg, Cog))
            continue
        ext = [(ex, ed, _prep(ex, math), _prep(ed, math)) for ex, ed in extra]
        # filter gradient
        idx = _samples(dw.shape, rng)
        g_, ref, emu, sc = [], [], [], []
        for co, ci, kh, kw in idx:
            g, cs, os_ = grp_of(co)
            j = (co - g * Cog, ci, kh, kw)
            wsh = (Cog, Cg, w.shape[2], w.shape[3])
            g_.append(dw[co, ci, kh, kw])
            r_, e_, s_ = 0.0, 0.0, 0.0
            for xx, dd, xxp, ddp in [(x, dy, xp, dyp)] + ext:
                r_ += oracle.conv_bwd_filter_at(xx[:, cs], dd[:, os_], wsh, S, P, j)
                e_ += _emu(oracle.conv_bwd_filter_at, _sl(xxp, slice(None), cs),
                           _sl(ddp, slice(None), os_), math, wsh, S, P, j)
                s_ += oracle.conv_bwd_filter_at_abs(xx[:, cs], dd[:, os_], wsh, S, P, j)
            ref.append(r_)
            emu.append(e_)
            sc.append(s_)
        _check("dw", g_, ref, emu, sc, exact, math, f"{name} dW")
        # bias gradient in full (the oracle's plain sum over n, ho, wo)
        ref = oracle.conv_db(dy) + sum(oracle.conv_db(ed) for _, ed in extra)
        if exact:
            np.testing.assert_array_equal(np.asarray(db, np.float64), ref, err_msg=f"{name} db")
        else:
            scale = sum(np.abs(d_.astype(np.float64)).sum(axis=(0, 2, 3)) for d_ in [dy] + [e for _, e in extra])
            assert np.all(np.abs(np.asarray(db, np.float64) - ref) <= 1e-5 * scale + 1e-30), name
        dx_terms.append((w, wp, dy, dyp, Cg, Cog))
    if "dx" not in u["arrays"]:
        assert u["data_fed"]   # the data-fed first layer has no backward-data pass (R9)
        return
    dx = _load(tmp, i, "dx")
    idx = _samples(dx.shape, rng)
    g_, ref, emu, sc = [], [], [], []
    for n, ci, h, ww in idx:
        rr = ee = ss = 0.0
        for w, wp, dy, dyp, Cg, Cog in dx_terms:
            g = ci // Cg
            os_ = slice(g * Cog, (g + 1) * Cog)
            j = (0, ci - g * Cg, h, ww)
            xs = (1, Cg) + tuple(dx.shape[2:])
            rr += oracle.conv_bwd_data_at(dy[n:n + 1, os_], w[os_], xs, S, P, j)
            ee += _emu(oracle.conv_bwd_data_at, _sl(dyp, slice(n, n + 1), os_), _sl(wp, os_), math,
                       xs, S, P, j)
            ss += oracle.conv_bwd_data_at(dy[n:n + 1, os_], w[os_], xs, S, P, j, absmode=True)
        g_.append(dx[n, ci, h, ww])
        ref.append(rr)
        emu.append(ee)
        sc.append(ss)
    _check("dx", g_, ref, emu, sc, exact, math, f"{'+'.join(u['names'])} dx")


CASES = [(1, "bf16", False), (2, "bf16", False), (3, "bf16", False), (4, "bf16", False),
         (4, "tf32", False), (5, "bf16", False), (5, "bf16", True), (6, "bf16", False),
         (7, "bf16", True),
         (1, "fp32", False), (2, "fp32", False), (3, "fp32", False), (4, "fp32", False),
         (5, "fp32", False), (6, "fp32", False), (7, "fp32", True), (7, "fp32", False),
         (8, "bf16", True), (8, "fp32", False), (9, "fp32", False), (9, "bf16", True)]


@pytest.mark.parametrize("case", CASES, ids=lambda c: f"cfg{c[0]}-{c[1]}-{'exact' if c[2] else 'float'}")
def test_fullsize_sampled_parity(case, tmp_path):
    workload, math, exact = case
    meta = _bench_dump(tmp_path, workload, math, exact)
    assert meta["workload"] == workload and meta["math"] == math
    rng = np.random.Generator(np.random.PCG64(1000 + workload))
    units = meta["units"]
    for i, u in enumerate(units):
        extra = [(np.asarray(_load(tmp_path, j, "x")), np.asarray(_load(tmp_path, j, "dy")))
                 for j, v in enumerate(units) if v.get("shares") == u["names"][0]]
        _check_unit(tmp_path, i, u, math, exact, rng, extra)


def test_fullsize_whole_tensor_exact(tmp_path):
    """CaffeNet conv1-5, batch 256, integer data: bench.py's own plans and graph-replayed step in
    bf16, tf32 and fp32 (3xTF32); every output tensor (y, dx, dW, db of every layer) equals the
    whole-tensor oracle bit for bit in every mode."""
    metas = {m: _bench_dump(tmp_path / m, 4, m, True) for m in ("bf16", "tf32", "fp32")}
    units = metas["bf16"]["units"]
    for i, u in enumerate(units):
        S, P = u["S"], u["P"]
        x = np.asarray(_load(tmp_path / "bf16", i, "x"))
        w = np.asarray(_load(tmp_path / "bf16", i, "w"))
        b = np.asarray(_load(tmp_path / "bf16", i, "b"))
        dy = np.asarray(_load(tmp_path / "bf16", i, "dy"))
        for m in ("tf32", "fp32"):   # the same integer draws in every mode
            for k, v in (("x", x), ("w", w), ("dy", dy)):
                np.testing.assert_array_equal(np.asarray(_load(tmp_path / m, i, k)), v)
        ref = {"y": oracle.conv_fwd(x, w, b, S, P)}
        ref["dw"], ref["db"] = oracle.conv_bwd_filter(x, dy, w.shape, S, P)
        if not u["data_fed"]:
            ref["dx"] = oracle.conv_bwd_data(dy, w, x.shape, S, P)
        for m in ("bf16", "tf32", "fp32"):
            for k, r in ref.items():
                np.testing.assert_array_equal(np.asarray(_load(tmp_path / m, i, k)),
                                              r.astype(np.float32), err_msg=f"{m} {u['names'][0]} {k}")
