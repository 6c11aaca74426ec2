"""Diagnostic: per-CTA cycle split of the igemm issue warps (GLP_DEBUG_CLK): MMA-warp loop
total, its waits on `full` (data not ready) and `tempty` (epilogue behind), producer waits on
`empty` (ring full).  Usage: python tools/clk_probe.py layer:pass ...
Needs the diagnostic library (the product libglp.so has no such hooks):
    python -m paper_conf_icpp_futhys18_b200._build --diag
    GLP_LIB=paper_conf_icpp_futhys18_b200/libglp_diag.so python tools/clk_probe.py ..."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
dev = torch.device("cuda:0")
buf = torch.zeros(4 * 1024, dtype=torch.int64, device=dev)
os.environ["GLP_DEBUG_CLK"] = str(buf.data_ptr())
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import config, gen_layer
layers = {l.name: l for l in config(4)}
for spec in sys.argv[1:]:
    name, passname = spec.split(":")
    l = layers[name]
    d = gen_layer(l)
    t = {k: torch.from_numpy(v).to(dev) for k, v in d.items()}
    L = glp.ConvLayer(l.N, l.C, l.H, l.W, l.Co, l.K, l.S, l.P, math=os.environ.get("MATH", "bf16"))
    y = torch.empty(L.y_shape, device=dev); dx = torch.empty(L.x_shape, device=dev)
    L.stage_pack(glp.GLP_PACK_X, t["x"]); L.stage_pack(glp.GLP_PACK_DY, t["dy"])
    L.stage_pack(glp.GLP_PACK_W_FWD if passname == "fwd" else glp.GLP_PACK_W_BWD_DATA, t["w"])
    f = {"fwd": lambda: L.stage_fwd(t["b"], y), "bwd_data": lambda: L.stage_bwd_data(dx),
         "bwd_filter": lambda: L.stage_bwd_filter()}[passname]
    for _ in range(3): f()
    buf.zero_()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); f(); e1.record(); torch.cuda.synchronize()
    c = buf.view(-1, 4).cpu().numpy()
    grid = int((c[:, 0] > 0).sum() + (c[:, 3] > 0).sum()) if False else None
    ep = c[len(c) // 2:] if False else None
    act = c[c[:, 0] > 0]
    prod = c[:, 3][c[:, 3] > 0]
    tot = act[:, 0].mean()
    print(f"{spec:28s} {e0.elapsed_time(e1)*1e3:7.1f}us  mma-loop {tot:9.0f} cyc  wait-full {act[:,1].mean()/tot:5.1%}"
          f"  wait-tempty {act[:,2].mean()/tot:5.1%}  producer wait-empty {prod.mean()/tot if len(prod) else 0:5.1%}"
          f"  (MMA CTAs {len(act)})", flush=True)
    g = L.info.grid_fwd if passname == "fwd" else (L.info.grid_bwd_data if passname == "bwd_data" else L.info.grid_bwd_filter)
    e = c[g:2 * g]
    e = e[e[:, 0] > 0]
    if len(e):
        print(f"{'':28s} epilogue warp0: loop {e[:,0].mean():9.0f} cyc  wait-tfull {e[:,1].mean()/e[:,0].mean():5.1%}"
              f"  tmem-ld {e[:,2].mean()/e[:,0].mean():5.1%}  tiles {e[:,3].mean():.1f}"
              f"  -> {(e[:,0].mean()-e[:,1].mean())/max(1,e[:,3].mean()):.0f} busy cyc/tile", flush=True)
