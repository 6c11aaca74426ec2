"""Probe: filter-gradient parity with CTA pairs (GLP_WGRAD_CG2=1) on integer data (exact), with a
map of which dW rows (ci, tap) / columns (co) are wrong (diagnostic)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import gen_custom
dev = torch.device("cuda:0")
shapes = [(2, 64, 8, 8, 128, 3, 1, 1), (2, 64, 8, 8, 256, 3, 1, 1), (2, 128, 8, 8, 128, 1, 1, 0),
          (2, 96, 9, 9, 256, 5, 1, 2)]
for cg in (os.environ.get("CGS", "0 1").split()):
    os.environ["GLP_WGRAD_CG2"] = cg
    for math in ("bf16", "tf32"):
        for (N, C, H, W, Co, K, S, P) in shapes:
            Ho = oracle.out_dim(H, K, S, P)
            d = gen_custom(N, C, H, W, Co, K, K, 5, exact=True, Ho=Ho, Wo=Ho)
            L = glp.ConvLayer(N, C, H, W, Co, K, S, P, math=math)
            t = {k: torch.from_numpy(v).to(dev) for k, v in d.items()}
            dw = torch.full(L.w_shape, float("nan"), device=dev)
            L.bwd_filter(t["x"], t["dy"], dw, None)
            torch.cuda.synchronize()
            rdw, _ = oracle.conv_bwd_filter(d["x"], d["dy"], d["w"].shape, S, P, with_bias=False)
            g = dw.cpu().numpy()
            bad = ~np.isclose(g, rdw, rtol=0, atol=0)
            msg = f"cg2={cg} {math} {(C, Co, K)} bn={L.info.tile_n_bwd_filter} bad={bad.mean():.3f}"
            if bad.any():
                co_bad = np.where(bad.any(axis=(1, 2, 3)))[0]
                ci_bad = np.where(bad.any(axis=(0, 2, 3)))[0]
                msg += f" co[{co_bad.min()}..{co_bad.max()}] n={len(co_bad)} ci[{ci_bad.min()}..{ci_bad.max()}] n={len(ci_bad)}"
                msg += f" nan={np.isnan(g).mean():.3f}"
                i = np.argwhere(bad)[0]
                msg += f" first={tuple(i)} got={g[tuple(i)]} ref={rdw[tuple(i)]}"
            print(msg, flush=True)
