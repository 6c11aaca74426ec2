"""Probe: wgrad/fwd/dgrad parity per shape with CTA pairs on/off (diagnostic)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import gen_custom
dev = torch.device("cuda:0")
shapes = [(4, 64, 8, 8, 128, 3, 1, 1), (4, 64, 8, 8, 256, 3, 1, 1), (4, 32, 8, 8, 64, 3, 1, 1),
          (4, 128, 16, 16, 128, 1, 1, 0), (4, 20, 12, 12, 50, 5, 1, 2)]
for cg in ("1", "2"):
    os.environ["GLP_CTA_GROUP"] = cg
    for math in ("bf16", "tf32"):
        for (N, C, H, W, Co, K, S, P) in shapes:
            Ho = oracle.out_dim(H, K, S, P)
            d = gen_custom(N, C, H, W, Co, K, K, 5, exact=True, Ho=Ho, Wo=Ho)
            L = glp.ConvLayer(N, C, H, W, Co, K, S, P, math=math)
            t = {k: torch.from_numpy(v).to(dev) for k, v in d.items()}
            dw = torch.full(L.w_shape, float("nan"), device=dev)
            y = torch.full(L.y_shape, float("nan"), device=dev)
            L.fwd(t["x"], t["w"], t["b"], y)
            L.bwd_filter(t["x"], t["dy"], dw, None)
            torch.cuda.synchronize()
            rdw, _ = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, S, P, with_bias=False)
            ry = oracle.conv_fwd(d["x"], d["w"], d["b"], S, P)
            ew = oracle.normwise_err(dw.cpu().numpy(), rdw)
            ey = oracle.normwise_err(y.cpu().numpy(), ry)
            ka = L.kernel_attr(2)
            print(f"cg={cg} {math} {(C, Co, K)} wgrad err={ew:.3g} fwd err={ey:.3g} "
                  f"bn_w={L.info.tile_n_bwd_filter} splits={L.info.splits_wgrad}", flush=True)
