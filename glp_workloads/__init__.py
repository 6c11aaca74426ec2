"""Seeded synthetic workloads shared by the CUDA path's tests/bench and the oracle.

Holds ONLY shapes (Table 5, P334-355, at the BASELINE.json batch sizes) and the
random-number recipe of DESIGN.md §Inputs; none of the method's arithmetic.
Both sides receive the same bytes from these generators.

Recipe (numpy ``Generator(PCG64(seed))``, seed = 0x474C5034 + 1000*cfg + 10*layer + tensor,
tensor: x=0, W=1, b=2, dy=3):
  data-fed x ~ U[0,1)            (pixel intensities)
  inner x    ~ max(0, N(0,1))    (post-ReLU activations, ~50% zeros)
  W          ~ U[-a, a], a = sqrt(3 / (C_i*K_h*K_w))   (Caffe "xavier", fan-in)
  b          ~ U[-0.1, 0.1]
  dy         ~ N(0,1) / N_global (batch-averaged loss)
  exact-arithmetic variant: integers, x/W/dy in [-2,2] (data layer x in [0,2]), b in [-4,4].
"""
from __future__ import annotations

from dataclasses import dataclass, replace
from typing import Dict, List

import numpy as np

SEED_BASE = 0x474C5034


@dataclass(frozen=True)
class Layer:
    name: str
    N: int
    C: int
    H: int
    W: int
    Co: int
    K: int
    S: int
    P: int
    Ho: int            # literal from Table 5 geometry (checked against oracle.out_dim in tests)
    data_fed: bool     # bottom is the data layer -> benchmark skips dgrad (R9)
    cfg: int = 0
    index: int = 0
    groups: int = 1    # Caffe convolution groups (CaffeNet conv2/4/5 use 2; Table 5 lists 1)

    @property
    def x_shape(self):
        return (self.N, self.C, self.H, self.W)

    @property
    def w_shape(self):
        return (self.Co, self.C // self.groups, self.K, self.K)

    @property
    def y_shape(self):
        return (self.N, self.Co, self.Ho, self.Ho)

    def with_batch(self, n: int) -> "Layer":
        return replace(self, N=int(n))

    def flops_per_pass(self) -> float:
        """2*C_o*C_i*K_h*K_w*H_o*W_o per image, times N (C_i per group)."""
        return 2.0 * self.Co * (self.C // self.groups) * self.K * self.K * self.Ho * self.Ho * self.N


def _L(name, N, C, HW, Co, K, S, P, Ho, data_fed, groups=1):
    return Layer(name, N, C, HW, HW, Co, K, S, P, Ho, data_fed, groups=groups)


# Table 5 (P334-355).  LeNet = the Siamese conv1/conv2 shapes (R20).
_TABLE: Dict[int, List[Layer]] = {
    1: [_L("lenet_conv1", 64, 1, 28, 20, 5, 1, 0, 24, True)],
    2: [_L("lenet_conv1", 64, 1, 28, 20, 5, 1, 0, 24, True),
        _L("lenet_conv2", 64, 20, 12, 50, 5, 1, 0, 8, False)],
    3: [_L("cifar10_conv1", 100, 3, 32, 32, 5, 1, 2, 32, True),
        _L("cifar10_conv2", 100, 32, 16, 32, 5, 1, 2, 16, False),
        _L("cifar10_conv3", 100, 32, 8, 64, 5, 1, 2, 8, False)],
    4: [_L("caffenet_conv1", 256, 3, 227, 96, 11, 4, 0, 55, True),
        _L("caffenet_conv2", 256, 96, 27, 256, 5, 1, 2, 27, False),
        _L("caffenet_conv3", 256, 256, 13, 384, 3, 1, 1, 13, False),
        _L("caffenet_conv4", 256, 384, 13, 384, 3, 1, 1, 13, False),
        _L("caffenet_conv5", 256, 384, 13, 256, 3, 1, 1, 13, False)],
    # GoogLeNet Table 5 units at the BASELINE batch 128 (R19); inputs synthesised
    # at the units' own 7x7 shapes.  None is fed by the data layer.
    5: [_L("googlenet_conv_1", 128, 160, 7, 320, 3, 1, 1, 7, False),
        _L("googlenet_conv_2", 128, 832, 7, 32, 1, 1, 0, 7, False),
        _L("googlenet_conv_3", 128, 832, 7, 384, 1, 1, 0, 7, False),
        _L("googlenet_conv_4", 128, 192, 7, 384, 3, 1, 1, 7, False),
        _L("googlenet_conv_5", 128, 832, 7, 192, 1, 1, 0, 7, False),
        _L("googlenet_conv_6", 128, 832, 7, 48, 1, 1, 0, 7, False)],
    # the complete inception 5a and 5b modules (all 12 convolutions; branch
    # widths from the GoogLeNet prototxt [ext], Table 5 covers 6 of them: conv_1 = 5a/3x3,
    # conv_2 = 5a/5x5_reduce, conv_3 = 5b/1x1, conv_4 = 5b/3x3, conv_5 = 5b/3x3_reduce,
    # conv_6 = 5b/5x5_reduce), batch 128, 7x7 maps.  pool_proj reads the 3x3 max-pool of the
    # module input (same 832x7x7 shape; synthesised).
    6: [_L("i5a_1x1", 128, 832, 7, 256, 1, 1, 0, 7, False),
        _L("i5a_3x3_reduce", 128, 832, 7, 160, 1, 1, 0, 7, False),
        _L("i5a_5x5_reduce", 128, 832, 7, 32, 1, 1, 0, 7, False),
        _L("i5a_3x3", 128, 160, 7, 320, 3, 1, 1, 7, False),
        _L("i5a_5x5", 128, 32, 7, 128, 5, 1, 2, 7, False),
        _L("i5a_pool_proj", 128, 832, 7, 128, 1, 1, 0, 7, False),
        _L("i5b_1x1", 128, 832, 7, 384, 1, 1, 0, 7, False),
        _L("i5b_3x3_reduce", 128, 832, 7, 192, 1, 1, 0, 7, False),
        _L("i5b_5x5_reduce", 128, 832, 7, 48, 1, 1, 0, 7, False),
        _L("i5b_3x3", 128, 192, 7, 384, 3, 1, 1, 7, False),
        _L("i5b_5x5", 128, 48, 7, 128, 5, 1, 2, 7, False),
        _L("i5b_pool_proj", 128, 832, 7, 128, 1, 1, 0, 7, False)],
    # CaffeNet as the Caffe model defines it, with group = 2 on conv2, conv4
    # and conv5 [ext: bvlc_reference_caffenet]; Table 5 (P345-349) lists the full C_i (R4).
    7: [_L("caffenet_conv1", 256, 3, 227, 96, 11, 4, 0, 55, True),
        _L("caffenet_conv2_g2", 256, 96, 27, 256, 5, 1, 2, 27, False, groups=2),
        _L("caffenet_conv3", 256, 256, 13, 384, 3, 1, 1, 13, False),
        _L("caffenet_conv4_g2", 256, 384, 13, 384, 3, 1, 1, 13, False, groups=2),
        _L("caffenet_conv5_g2", 256, 384, 13, 256, 3, 1, 1, 13, False, groups=2)],
}


# the Siamese network of Table 5 (P341-344) with its shared weights: the two
# towers (conv1, conv2) and (conv1_p, conv2_p) read different images but conv1_p / conv2_p use
# conv1's / conv2's parameters [ext: Caffe mnist_siamese, param names shared], so their filter
# gradients accumulate into one diff (Caffe beta = 1; glp_conv_bwd_filter accumulate = 1).  The
# sharing towers are listed first so that, visited in reverse for the backward, every owner's
# gradient overwrites before its sharer accumulates.
_TABLE[8] = [_L("siamese_conv1_p", 64, 1, 28, 20, 5, 1, 0, 24, True),
             _L("siamese_conv2_p", 64, 20, 12, 50, 5, 1, 0, 8, False),
             _L("siamese_conv1", 64, 1, 28, 20, 5, 1, 0, 24, True),
             _L("siamese_conv2", 64, 20, 12, 50, 5, 1, 0, 8, False)]

# GoogLeNet's whole convolution stack at 224 x 224, batch 128 (BASELINE.json
# configs[4] "synthetic 3x224x224"): conv1 7x7/2, conv2_reduce, conv2 and the nine inception
# modules (3a-5b: 1x1, 3x3_reduce, 3x3, 5x5_reduce, 5x5, pool_proj) -- 57 convolutions, branch
# widths from the GoogLeNet prototxt [ext: Szegedy et al. 2015, Table 1]; Table 5 lists 6 of them
# (P350-355).  Each layer's input is synthesised at its own shape (pooling / concatenation are not
# on the path).
_INCEPTION = [  # name, H = W, C_in, [1x1, 3x3_reduce, 3x3, 5x5_reduce, 5x5, pool_proj]
    ("3a", 28, 192, [64, 96, 128, 16, 32, 32]), ("3b", 28, 256, [128, 128, 192, 32, 96, 64]),
    ("4a", 14, 480, [192, 96, 208, 16, 48, 64]), ("4b", 14, 512, [160, 112, 224, 24, 64, 64]),
    ("4c", 14, 512, [128, 128, 256, 24, 64, 64]), ("4d", 14, 512, [112, 144, 288, 32, 64, 64]),
    ("4e", 14, 528, [256, 160, 320, 32, 128, 128]), ("5a", 7, 832, [256, 160, 320, 32, 128, 128]),
    ("5b", 7, 832, [384, 192, 384, 48, 128, 128])]


def _googlenet_full(N=128):
    ls = [_L("g_conv1_7x7_s2", N, 3, 224, 64, 7, 2, 3, 112, True),
          _L("g_conv2_reduce", N, 64, 56, 64, 1, 1, 0, 56, False),
          _L("g_conv2_3x3", N, 64, 56, 192, 3, 1, 1, 56, False)]
    for m, hw, cin, (a, b, c, d, e, f) in _INCEPTION:
        ls += [_L(f"g_{m}_1x1", N, cin, hw, a, 1, 1, 0, hw, False),
               _L(f"g_{m}_3x3_reduce", N, cin, hw, b, 1, 1, 0, hw, False),
               _L(f"g_{m}_5x5_reduce", N, cin, hw, d, 1, 1, 0, hw, False),
               _L(f"g_{m}_pool_proj", N, cin, hw, f, 1, 1, 0, hw, False),
               _L(f"g_{m}_3x3", N, b, hw, c, 3, 1, 1, hw, False),
               _L(f"g_{m}_5x5", N, d, hw, e, 5, 1, 2, hw, False)]
    return ls


_TABLE[9] = _googlenet_full()

# Shared-parameter layers: sharer -> owner (same W and b; the sharer's filter gradient is added
# to the owner's with accumulate = 1 after the owner's own).
SHARED: Dict[int, Dict[str, str]] = {
    8: {"siamese_conv1_p": "siamese_conv1", "siamese_conv2_p": "siamese_conv2"},
}

# Sibling layers that read the same input tensor in the real network and can run as one fused
# group (include/glp.h "fused sibling groups"): GoogLeNet inception 5b's
# 1x1, 3x3_reduce and 5x5_reduce branches (Table 5 conv_3, conv_5, conv_6) all read 5b's
# 832-channel input.  The group uses the first member's x draw as the shared input.
SIBLINGS: Dict[int, List[List[str]]] = {
    5: [["googlenet_conv_3", "googlenet_conv_5", "googlenet_conv_6"]],
    6: [["i5a_1x1", "i5a_3x3_reduce", "i5a_5x5_reduce"],
        ["i5b_1x1", "i5b_3x3_reduce", "i5b_5x5_reduce"]],
    9: [[f"g_{m}_1x1", f"g_{m}_3x3_reduce", f"g_{m}_5x5_reduce"] for m, *_ in _INCEPTION],
}

# The network DAG of a workload as levels of layers that are independent of each other in the
# real network (same level = may run concurrently; level l+1 depends on level l).  Workloads not
# listed are chains.  GoogLeNet (5): conv_1 (5a/3x3, fed by 5a/3x3_reduce) and conv_2
# (5a/5x5_reduce) are parallel branches of module 5a; the 5b reduce/1x1 branches read 5a's output;
# conv_4 (5b/3x3) reads 5b/3x3_reduce.  Inception 5a+5b (6): per module, the branches that read
# the module input (1x1, 3x3_reduce, 5x5_reduce, pool_proj after the max-pool), then the 3x3 and
# 5x5 convolutions of the reduced maps.
LEVELS: Dict[int, List[List[str]]] = {
    # Siamese: the two towers run side by side (conv2 reads conv1's output in each tower)
    8: [["siamese_conv1_p", "siamese_conv1"], ["siamese_conv2_p", "siamese_conv2"]],
    # full GoogLeNet: the stem is a chain; per module, the branches that read the module input,
    # then the 3x3 and 5x5 convolutions of the reduced maps
    9: [["g_conv1_7x7_s2"], ["g_conv2_reduce"], ["g_conv2_3x3"]] +
       [lv for m, *_ in _INCEPTION
        for lv in ([f"g_{m}_1x1", f"g_{m}_3x3_reduce", f"g_{m}_5x5_reduce", f"g_{m}_pool_proj"],
                   [f"g_{m}_3x3", f"g_{m}_5x5"])],
    5: [["googlenet_conv_1", "googlenet_conv_2"],
        ["googlenet_conv_3", "googlenet_conv_5", "googlenet_conv_6"],
        ["googlenet_conv_4"]],
    6: [["i5a_1x1", "i5a_3x3_reduce", "i5a_5x5_reduce", "i5a_pool_proj"],
        ["i5a_3x3", "i5a_5x5"],
        ["i5b_1x1", "i5b_3x3_reduce", "i5b_5x5_reduce", "i5b_pool_proj"],
        ["i5b_3x3", "i5b_5x5"]],
}

CONFIG_NAMES = {
    1: "lenet_conv1_b64",
    2: "lenet5_conv_stack_b64",
    3: "cifar10_quick_conv_b100",
    4: "caffenet_conv1-5_b256",
    5: "googlenet_table5_units_b128",
    6: "googlenet_inception_5a5b_b128",
    7: "caffenet_group2_conv1-5_b256",
    8: "siamese_lenet_shared_b64",
    9: "googlenet_full_224_b128",
}


def config(cfg: int) -> List[Layer]:
    return [replace(l, cfg=cfg, index=i) for i, l in enumerate(_TABLE[cfg])]


def all_layers() -> List[Layer]:
    out = []
    for c in sorted(_TABLE):
        out.extend(config(c))
    return out


def seed(cfg: int, layer: int, tensor: int) -> int:
    return SEED_BASE + 1000 * cfg + 10 * layer + tensor


def _rng(cfg, layer, tensor):
    return np.random.Generator(np.random.PCG64(seed(cfg, layer, tensor)))


def gen_layer(layer: Layer, n_global: int = None, exact: bool = False, batch: int = None):
    """Return dict(x, w, b, dy) of float32 numpy arrays for one layer (same bytes for both sides).

    ``batch`` overrides N (samples are the first ``batch`` of the stream's draws order)."""
    N = layer.N if batch is None else int(batch)
    n_global = N if n_global is None else n_global
    c, i = layer.cfg, layer.index
    xs = (N, layer.C, layer.H, layer.W)
    ws = layer.w_shape
    ys = (N, layer.Co, layer.Ho, layer.Ho)
    if exact:
        lo = 0 if layer.data_fed else -2
        x = _rng(c, i, 0).integers(lo, 3, size=xs).astype(np.float32)
        w = _rng(c, i, 1).integers(-2, 3, size=ws).astype(np.float32)
        b = _rng(c, i, 2).integers(-4, 5, size=(layer.Co,)).astype(np.float32)
        dy = _rng(c, i, 3).integers(-2, 3, size=ys).astype(np.float32)
    else:
        if layer.data_fed:
            x = _rng(c, i, 0).random(xs, dtype=np.float32)
        else:
            x = np.maximum(_rng(c, i, 0).standard_normal(xs, dtype=np.float32), 0.0)
        a = np.float32(np.sqrt(3.0 / (layer.C // layer.groups * layer.K * layer.K)))
        w = _rng(c, i, 1).uniform(-a, a, size=ws).astype(np.float32)
        b = _rng(c, i, 2).uniform(-0.1, 0.1, size=(layer.Co,)).astype(np.float32)
        dy = (_rng(c, i, 3).standard_normal(ys, dtype=np.float32) / np.float32(n_global)).astype(np.float32)
    return {"x": np.ascontiguousarray(x), "w": np.ascontiguousarray(w),
            "b": np.ascontiguousarray(b), "dy": np.ascontiguousarray(dy)}


def gen_custom(N, C, H, W, Co, Kh, Kw, seed_: int, exact: bool = False, Ho=None, Wo=None,
               data_fed: bool = False):
    """Generator for ad-hoc shapes (odd strides/pads, ragged tails).  Ho/Wo are supplied by
    the caller (the generator holds no conv arithmetic)."""
    r = np.random.Generator(np.random.PCG64(int(seed_)))
    xs, ws, ys = (N, C, H, W), (Co, C, Kh, Kw), (N, Co, Ho, Wo)
    if exact:
        x = r.integers(0 if data_fed else -2, 3, size=xs).astype(np.float32)
        w = r.integers(-2, 3, size=ws).astype(np.float32)
        b = r.integers(-4, 5, size=(Co,)).astype(np.float32)
        dy = r.integers(-2, 3, size=ys).astype(np.float32)
    else:
        x = r.standard_normal(xs, dtype=np.float32)
        a = np.float32(np.sqrt(3.0 / max(1, C * Kh * Kw)))
        w = r.uniform(-a, a, size=ws).astype(np.float32)
        b = r.uniform(-0.1, 0.1, size=(Co,)).astype(np.float32)
        dy = (r.standard_normal(ys, dtype=np.float32) / np.float32(max(N, 1))).astype(np.float32)
    return {"x": x, "w": w, "b": b, "dy": dy}
