"""A/B timing of one layer-pass GEMM stage under plan-option variants (CUDA events, warm).
usage: python tools/pass_time.py caffenet_conv1:bwd_filter fp32 '{}' '{"wgrad_tile_n":128}' ...
Prints the average stage time (GEMM only; packs excluded) and the plan info of each variant."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import config, gen_layer

dev = torch.device("cuda:0")
name, passname = sys.argv[1].split(":")
math = sys.argv[2]
wl = int(os.environ.get("WL", "4"))
l = {x.name: x for x in config(wl)}[name]
t = {k: torch.from_numpy(v).to(dev) for k, v in gen_layer(l).items()}
for spec in sys.argv[3:]:
    opts = json.loads(spec)
    L = glp.ConvLayer(l.N, l.C, l.H, l.W, l.Co, l.K, l.S, l.P, math=math, options=opts or None)
    y = torch.empty(L.y_shape, device=dev); dx = torch.empty(L.x_shape, device=dev)
    dw = torch.empty(L.w_shape, device=dev); db = torch.empty(l.Co, device=dev)
    L.stage_pack(glp.GLP_PACK_X, t["x"]); L.stage_pack(glp.GLP_PACK_W_FWD, t["w"])
    L.stage_pack(glp.GLP_PACK_DY_DB, t["dy"]); L.stage_pack(glp.GLP_PACK_W_BWD_DATA, t["w"])
    run = {"fwd": lambda: L.stage_fwd(t["b"], y), "bwd_data": lambda: L.stage_bwd_data(dx),
           "bwd_filter": lambda: L.stage_bwd_filter()}[passname]
    for _ in range(3):
        run()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(10):
        run()
    e1.record()
    torch.cuda.synchronize()
    i = L.info
    print(f"{spec:40s} {e0.elapsed_time(e1) / 10 * 1e3:9.1f} us  tile_n {i.tile_n_fwd}/{i.tile_n_bwd_data}/"
          f"{i.tile_n_bwd_filter} grid {i.grid_fwd}/{i.grid_bwd_data}/{i.grid_bwd_filter} "
          f"splits {i.splits_wgrad} stages {i.stages_fwd}/{i.stages_bwd_data}/{i.stages_bwd_filter}", flush=True)
