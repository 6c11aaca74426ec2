"""Diagnostic: print the plan summary (grid, tiles, stages, splits) of every layer of a config."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_icpp_futhys18_b200 as glp
from glp_workloads import config
for l in config(int(os.environ.get("WORKLOAD", "4"))):
    L = glp.ConvLayer(l.N, l.C, l.H, l.W, l.Co, l.K, l.S, l.P, math=os.environ.get("MATH", "bf16"))
    i = L.info
    print(f"{l.name:16s} grid {i.grid_fwd}/{i.grid_bwd_data}/{i.grid_bwd_filter} tiles {i.tiles_fwd}/"
          f"{i.tiles_bwd_data}/{i.tiles_bwd_filter} tn {i.tile_n_fwd}/{i.tile_n_bwd_data}/"
          f"{i.tile_n_bwd_filter} stages {i.stages_fwd}/{i.stages_bwd_data}/{i.stages_bwd_filter} "
          f"splits {i.splits_wgrad}")
