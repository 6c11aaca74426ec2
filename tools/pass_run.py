"""Diagnostic driver for ncu: run one layer-pass of a workload through the staged API.
usage: python tools/pass_run.py caffenet_conv1:bwd_filter [iters] [workload]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import config, gen_layer
dev = torch.device("cuda:0")
spec = sys.argv[1]
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 3
wl = int(sys.argv[3]) if len(sys.argv) > 3 else 4
name, passname = spec.split(":")
l = {x.name: x for x in config(wl)}[name]
t = {k: torch.from_numpy(v).to(dev) for k, v in gen_layer(l).items()}
L = glp.ConvLayer(l.N, l.C, l.H, l.W, l.Co, l.K, l.S, l.P, math=os.environ.get("MATH", "bf16"))
y = torch.empty(L.y_shape, device=dev); dx = torch.empty(L.x_shape, device=dev)
dw = torch.empty(L.w_shape, device=dev); db = torch.empty(l.Co, device=dev)
for _ in range(iters):
    if passname == "fwd":
        L.stage_pack(glp.GLP_PACK_X, t["x"]); L.stage_pack(glp.GLP_PACK_W_FWD, t["w"]); L.stage_fwd(t["b"], y)
    elif passname == "bwd_data":
        L.stage_pack(glp.GLP_PACK_DY, t["dy"]); L.stage_pack(glp.GLP_PACK_W_BWD_DATA, t["w"]); L.stage_bwd_data(dx)
    else:
        L.stage_pack(glp.GLP_PACK_X, t["x"]); L.stage_pack(glp.GLP_PACK_DY_DB, t["dy"])
        L.stage_bwd_filter(); L.stage_reduce(dw, db)
torch.cuda.synchronize()
print("ok", spec, L.info.as_dict())
