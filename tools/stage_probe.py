"""Diagnostic: time one GEMM stage with A loads / B loads / MMAs selectively skipped
(GLP_DEBUG_SKIP bits 0/1/2; results are garbage in the skipped modes).
Needs the diagnostic library (the product libglp.so has no such hooks):
    python -m paper_conf_icpp_futhys18_b200._build --diag
    GLP_LIB=paper_conf_icpp_futhys18_b200/libglp_diag.so python tools/stage_probe.py ..."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import config, gen_layer
dev = torch.device("cuda:0")
layers = {l.name: l for l in config(4)}
which = sys.argv[1:] or ["caffenet_conv3:fwd", "caffenet_conv2:fwd", "caffenet_conv2:bwd_data", "caffenet_conv3:bwd_filter"]
for spec in which:
    name, passname = spec.split(":")
    l = layers[name]
    d = gen_layer(l)
    t = {k: torch.from_numpy(v).to(dev) for k, v in d.items()}
    res = []
    for skip in [int(s) for s in os.environ.get("SKIPS", "0 1 2 3 4 7").split()]:
        os.environ["GLP_DEBUG_SKIP"] = str(skip)
        L = glp.ConvLayer(l.N, l.C, l.H, l.W, l.Co, l.K, l.S, l.P, math=os.environ.get("MATH", "bf16"))
        y = torch.empty(L.y_shape, device=dev); dx = torch.empty(L.x_shape, device=dev)
        L.stage_pack(glp.GLP_PACK_X, t["x"]); L.stage_pack(glp.GLP_PACK_DY, t["dy"])
        L.stage_pack(glp.GLP_PACK_W_FWD if passname == "fwd" else glp.GLP_PACK_W_BWD_DATA, t["w"])
        f = {"fwd": lambda: L.stage_fwd(t["b"], y), "bwd_data": lambda: L.stage_bwd_data(dx),
             "bwd_filter": lambda: L.stage_bwd_filter()}[passname]
        for _ in range(3): f()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20): f()
        e1.record(); torch.cuda.synchronize()
        res.append((skip, e0.elapsed_time(e1) / 20 * 1e3))
    fl = l.flops_per_pass()
    print(f"{spec:28s} " + "  ".join(f"skip{s}={us:7.1f}us" for s, us in res) + f"  full={fl/res[0][1]/1e6:.0f}TF/s", flush=True)
    os.environ.pop("GLP_DEBUG_SKIP")
