"""Calibration: torch reference rates for the pack-like memory patterns on this GPU (CUDA events).
fp32 -> bf16 contiguous cast, NCHW -> NHWC bf16 (torch permute+contiguous+cast), fp32 copy."""
import torch
dev = torch.device("cuda:0")


def t(fn, it=20):
    for _ in range(3):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(it):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / it * 1e3


for name, shape in [("conv1 dy", (256, 96, 55, 55)), ("conv2 dy", (256, 256, 27, 27)),
                    ("conv5 x", (256, 384, 13, 13)), ("conv1 x", (256, 3, 227, 227))]:
    x = torch.randn(shape, device=dev)
    nb = x.numel() * 4
    o = torch.empty(shape, device=dev, dtype=torch.bfloat16)
    us_cast = t(lambda: o.copy_(x))
    o2 = torch.empty((shape[0], shape[2], shape[3], shape[1]), device=dev, dtype=torch.bfloat16)
    us_perm = t(lambda: o2.copy_(x.permute(0, 2, 3, 1)))
    y = torch.empty_like(x)
    us_copy = t(lambda: y.copy_(x))
    print(f"{name:10s} {nb/1e6:7.1f} MB fp32: cast->bf16 {us_cast:7.1f} us ({nb*1.5/us_cast/1e3:5.0f} GB/s)"
          f"  nchw->nhwc bf16 {us_perm:7.1f} us ({nb*1.5/us_perm/1e3:5.0f} GB/s)"
          f"  fp32 copy {us_copy:7.1f} us ({nb*2/us_copy/1e3:5.0f} GB/s)")

# the library's packs, timed the same way (warm, back to back)
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import config
for l in config(4):
    L = glp.ConvLayer(l.N, l.C, l.H, l.W, l.Co, l.K, l.S, l.P, math="bf16")
    x = torch.randn(L.x_shape, device=dev)
    dy = torch.randn(L.y_shape, device=dev)
    us_x = t(lambda: L.stage_pack(glp.GLP_PACK_X, x))
    us_dy = t(lambda: L.stage_pack(glp.GLP_PACK_DY_DB, dy))
    bx, bdy = x.numel() * 4, dy.numel() * 4
    print(f"glp {l.name:16s} x pack {us_x:7.1f} us ({bx*1.5/us_x/1e3:5.0f} GB/s eq)   dy pack {us_dy:7.1f} us "
          f"({bdy*1.5/us_dy/1e3:5.0f} GB/s eq)")
