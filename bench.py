#!/usr/bin/env python
"""bench.py — conv-layer training throughput of the B200-native GLP4NN hot path.

Metric (BASELINE.json): conv fwd+bwd images/sec at 1/2/4/8 B200, with the dominant kernel's
fraction of the tensor-pipe roofline.  A step = one pass of the whole hot path over one batch:
for every conv layer of the workload, forward (pack x, pack W, tcgen05 implicit GEMM + bias),
then backward in reverse layer order (pack dy + db partials, backward-data GEMM — skipped for the
data-fed first layer, R9 — filter-gradient GEMM, fixed-order split reduction), then
(N > 1) one NCCL all_reduce(SUM) of the flat dW||db buffer.

Default workload: CaffeNet conv1-5 at batch 256 per GPU (BASELINE.json configs[3]; Table 5
P345-349), bf16 operands with fp32 accumulation.  The other configs are parity-test cases
(``--workload 1..5`` runs them too).

Launch: ``python bench.py --gpus N --steps K --warmup W``; for N > 1 under torchrun (one rank
per GPU, NCCL).  ``--impl reference`` times the fp64 CPU oracle (the reference arm of this tier).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from glp_workloads import CONFIG_NAMES, LEVELS, SHARED, SIBLINGS, config, gen_layer  # noqa: E402

METRIC = "conv fwd+bwd images/sec"
# the arithmetic each --math mode computes in (fp32 = 3xTF32 on tcgen05: fp32-accurate)
DTYPE = {"fp32": "fp32 (split: tf32 hi*hi + 2 bf16 cross terms; 3xtf32 on non-TMA layers)",
         "tf32": "tf32", "bf16": "bf16"}
UNIT = "images/s"
NOMINAL_TF32_OVER_BF16 = 1.1 / 2.25   # B200_PROFILING.md nominal dense ratio


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=100)
    p.add_argument("--warmup", type=int, default=10)
    p.add_argument("--impl", choices=["glp", "reference"], default="glp")
    p.add_argument("--workload", type=int, default=4, help="BASELINE.json config index 1..5")
    p.add_argument("--math", choices=["fp32", "bf16", "tf32"], default="fp32",
                   help="fp32 = 3xTF32 on tcgen05 (fp32-accurate, the paper's FP32 arithmetic)")
    p.add_argument("--scaling", choices=["weak", "strong"], default="strong",
                   help="strong (default, the BASELINE.json cfg4 wording): the config's global batch "
                        "sharded over the GPUs; weak: the config batch on every GPU")
    p.add_argument("--scheme", choices=["persistent", "pool"], default="persistent",
                   help="pool: the paper's prior-art scheme (per-sample kernels round-robin over a "
                        "stream pool sized by Eq. 7) as a comparator; 1 GPU")
    p.add_argument("--pool-streams", type=int, default=0,
                   help="stream-pool size (0 = the Eq. 7 bound)")
    p.add_argument("--exchange", choices=["nccl", "tree"], default="nccl",
                   help="tree: deterministic gradient exchange (filter gradients per batch leaf, "
                        "fixed binary tree over 8 leaves + recursive doubling; dW bitwise "
                        "identical for 1/2/4/8 GPUs); nccl: one all_reduce(SUM)")
    p.add_argument("--chain", action="store_true",
                   help="treat the workload as a chain of layers even where the network runs "
                        "branches in parallel (default: independent layers of a level run on "
                        "concurrent streams, glp_workloads.LEVELS)")
    p.add_argument("--no-fuse", action="store_true",
                   help="run sibling layers that share an input (GoogLeNet 5b 1x1 branches) as "
                        "separate layers instead of one fused group")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-extra-modes", action="store_true",
                   help="skip the bf16 / tf32 lines measured beside the fp32 headline (1 GPU)")
    p.add_argument("--dist-backend", choices=["nccl", "gloo"], default="nccl",
                   help="(tests) process-group backend; gloo + --same-device runs the N-rank step "
                        "on one GPU to exercise the multi-rank code path (timings meaningless)")
    p.add_argument("--same-device", action="store_true",
                   help="(tests) every rank on cuda:0 instead of cuda:LOCAL_RANK")
    p.add_argument("--dry-run", action="store_true",
                   help="(tests) launcher plumbing only: start the ranks, form a gloo process group "
                        "on CPU, all-reduce one tensor and print the line's n_gpus; no GPU work")
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--plan-options", default="",
                   help="JSON glp_plan_options_t fields for every plan (A/B runs of alternative "
                        "kernels/tilings; recorded in config)")
    p.add_argument("--e2e-steps", type=int, default=20)
    p.add_argument("--serial", action="store_true",
                   help="issue the step on one stream (default: the real-network stream DAG)")
    p.add_argument("--no-graph", action="store_true",
                   help="launch every step eagerly (default on 1 GPU: the step is captured once "
                        "into a CUDA graph and replayed)")
    p.add_argument("--exact-data", action="store_true",
                   help="(tests) integer-valued inputs (glp_workloads exact variant) instead of "
                        "the float recipe: every output is exact, so parity is bit for bit")
    p.add_argument("--dump", default=None,
                   help="(tests) after the timed steps, save every unit's inputs and outputs "
                        "(.npy) and a meta.json to this directory for full-size sampled parity")
    return p.parse_args()


# ------------------------------------------------------------------------- helpers ------------

def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def load_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return {"hbm_gbs": float(d["hbm_gbs"]), "bf16_tflops": float(d["bf16_tflops"]),
                "bf16_tflops_sustained": float(d.get("bf16_tflops_sustained", d["bf16_tflops"])),
                "source": "measured (MEASURED_PEAKS.json)"}
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
                "source": "fallback (B200_PROFILING.md)"}


class ClockSampler:
    """SM clocks and throttle reasons sampled DURING the timed region: an NVML thread polling every
    10 ms (starts immediately, so even a ~100 ms region gets samples); nvidia-smi -lms 200 as the
    fallback when NVML is unavailable."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")
    # NVML clocks-event reason bits (nvml.h nvmlClocksEventReason*)
    NVML_BITS = {"sw_power_cap": 0x4, "hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20,
                 "hw_thermal_slowdown": 0x40}

    def __init__(self, gpu_index):
        self.idx = gpu_index
        self.proc = None
        self.f = None
        self.thread = None
        self.samples = []
        self.mx = 0.0
        self.reasons = set()

    def _nvml_loop(self, h, nv):
        while not self.halt.is_set():
            try:
                self.samples.append(float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)))
                try:
                    bits = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                except AttributeError:
                    bits = nv.nvmlDeviceGetCurrentClocksThrottleReasons(h)
                for n, b in self.NVML_BITS.items():
                    if bits & b:
                        self.reasons.add(n)
            except Exception:
                pass
            self.halt.wait(0.01)

    def start(self):
        try:
            import threading
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.idx)
            self.mx = float(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM))
            self.halt = threading.Event()
            self.thread = threading.Thread(target=self._nvml_loop, args=(h, nv), daemon=True)
            self.thread.start()
            return
        except Exception:
            self.thread = None
        try:
            self.f = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.idx}", f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=self.f, stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.thread is not None:
            self.halt.set()
            self.thread.join(timeout=2)
            if not self.samples:
                return None
            return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.mx,
                    "reasons": sorted(self.reasons), "samples": len(self.samples), "source": "nvml"}
        if self.proc is None:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.f.flush()
        self.f.seek(0)
        rows = [l.strip().split(",") for l in self.f.read().splitlines() if l.strip()]
        os.unlink(self.f.name)
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            try:
                sm.append(float(r[0]))
                mx = max(mx, float(r[1]))
            except (ValueError, IndexError):
                continue
            for n, v in zip(names, r[3:7]):
                if v.strip().lower() == "active":
                    reasons.add(n)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm), "source": "nvidia-smi"}


# ------------------------------------------------------------------------- GLP arm ------------

PLAN_OPTIONS = {}   # --plan-options (A/B measurements of alternative plans; recorded in the line)


class LayerState:
    def __init__(self, layer, n_local, n_global, shard, math, dev, grads, idx, leaves=0):
        import torch
        import paper_conf_icpp_futhys18_b200 as glp
        self.glp = glp
        self.layer = layer
        self.name = layer.name
        self.n = n_local
        # leaves > 1: a leaf plan (the deterministic exchange: splits never cross a batch leaf)
        self.conv = glp.ConvLayer(n_local, layer.C, layer.H, layer.W, layer.Co, layer.K, layer.S,
                                  layer.P, math=math, device=dev.index, groups=layer.groups,
                                  options=dict(PLAN_OPTIONS, **({"wgrad_leaves": leaves} if leaves > 0 else {}))
                                  or None)
        if shard is None:
            d = gen_layer(layer, n_global=n_global, batch=n_local)
        else:  # strong scaling: this rank's contiguous slice of the global batch
            a, b = shard
            full = gen_layer(layer, n_global=n_global)
            d = {k: v for k, v in full.items()}
            d["x"] = full["x"][a:b].copy()
            d["dy"] = full["dy"][a:b].copy()
        self.host = {k: torch.from_numpy(v) for k, v in d.items()}
        self.t = {k: v.to(dev) for k, v in self.host.items()}
        self.y = torch.empty(self.conv.y_shape, device=dev)
        self.dx = None if layer.data_fed else torch.empty(self.conv.x_shape, device=dev)
        self.dw = grads.dw(idx)      # views into the flat dW||db buffer (one all_reduce per step)
        self.db = grads.db(idx)
        self.flops = float(self.layer.with_batch(n_local).flops_per_pass())
        self.leaves = None
        self.idx = idx
        # shared parameters (glp_workloads.SHARED): a sharer reads its owner's W and b and adds its
        # filter gradient to the owner's (accumulate = 1) after the owner's own
        self.owner = None
        self.has_sharer = False
        self.accumulate = False
        self.shared_keys = set()

    def share_params_of(self, owner):
        self.owner = owner
        owner.has_sharer = True
        self.accumulate = True
        for k in ("w", "b"):
            self.t[k] = owner.t[k]
            self.host[k] = owner.host[k]
        self.shared_keys = {"w", "b"}
        self.dw, self.db = owner.dw, owner.db

    def grad_idxs(self):
        """Slots of the flat dW||db buffer this unit writes (its all-reduce bucket)."""
        return [self.owner.idx if self.owner is not None else self.idx]

    def launches(self):
        """Kernels this unit launches per timed step: pack x, W pack(s), fwd GEMM, dy pack, dgrad
        GEMM, filter-gradient GEMM, dW and db reductions; a fused-dy plan (data-fed halo layer)
        launches no dy pack."""
        base = 9 if self.dx is not None else 7
        if self.dx is None and self.conv.info.wgrad_fused_dy:
            base -= 1
        return base

    # the step's kernel groups (one C call each; see step())
    def pack_x(self, st=None):
        self.conv.stage_pack(self.glp.GLP_PACK_X, self.t["x"], stream=st)

    def pack_w_fwd(self, st=None):
        self.conv.stage_pack(self.glp.GLP_PACK_W_FWD, self.t["w"], stream=st)

    def fwd(self, st=None):
        self.conv.stage_fwd(self.t["b"], self.y, stream=st)

    def pack_dy(self, st=None):
        self.conv.stage_pack(self.glp.GLP_PACK_DY_DB, self.t["dy"], stream=st)

    def pack_w_bwd(self, st=None):
        self.conv.stage_pack(self.glp.GLP_PACK_W_BWD_DATA, self.t["w"], stream=st)

    def bwd_data(self, st=None):
        self.conv.stage_bwd_data(self.dx, stream=st)

    def bwd_filter(self, st=None):
        self.conv.stage_bwd_filter(stream=st)

    def reduce(self, st=None):
        if self.leaves is None:
            self.conv.stage_reduce(self.dw, self.db, accumulate=self.accumulate, stream=st)
            return
        # deterministic exchange: one dW||db per leaf into the leaf buffers (the tree sums them)
        ex, sl = self.leaves, self.slot
        flat = ex.leaves.view(-1)
        self.conv.stage_reduce_leaves(flat[sl.w_off:], flat[sl.b_off:], ex.numel, stream=st)

    def host_inputs(self):
        return self.host, self.t


def kernel_name(states, rec):
    """The library kernel that ran a unit's pass (from the plan info: halo forms where chosen)."""
    for s in states:
        if s.name != rec["layer"]:
            continue
        info = s.conv.info
        if rec["pass"] == "fwd" and getattr(info, "fwd_halo", 0):
            return "hfwd_kernel"
        if rec["pass"] == "bwd_data" and getattr(info, "dgrad_halo", 0):
            return "hdgrad_kernel"
        if rec["pass"] == "bwd_filter" and getattr(info, "wgrad_halo", 0):
            return "hwgrad_kernel"
    return "igemm_kernel"


def set_exact_data(states):
    """--exact-data: every unit's inputs replaced by the integer variant of its seeded draws."""
    import torch
    for s in states:
        if isinstance(s, GroupState):
            ds = [gen_layer(m, exact=True, batch=s.n) for m in s.members]
            new = {"x": ds[0]["x"]}
            for i, d in enumerate(ds):
                for k in ("w", "b", "dy"):
                    new[f"{k}{i}"] = d[k]
        else:
            new = gen_layer(s.layer, exact=True, batch=s.n)
        for k, v in new.items():
            if k in s.shared_keys:   # the owner's parameters (replaced with the owner's draws)
                continue
            s.host[k] = torch.from_numpy(v)
            s.t[k].copy_(s.host[k])


def dump_units(states, path, workload, math):
    """--dump: the inputs and outputs of every unit after the timed steps (the launch
    configuration the bench measured) for tests/test_gpu_fullsize.py."""
    import numpy as np
    import torch
    torch.cuda.synchronize()
    os.makedirs(path, exist_ok=True)
    meta = {"workload": workload, "math": math, "units": []}
    for i, s in enumerate(states):
        grp = isinstance(s, GroupState)
        l = s.layer
        u = {"kind": "group" if grp else "layer",
             "names": [m.name for m in s.members] if grp else [l.name],
             "N": s.n, "C": l.C, "H": l.H, "W": l.W, "K": l.K, "S": l.S, "P": l.P,
             "groups": l.groups, "data_fed": l.data_fed,
             "Co": [m.Co for m in s.members] if grp else [l.Co],
             "shares": None if s.owner is None else s.owner.name}
        arrays = {k: v.cpu().numpy() for k, v in s.t.items()}
        if grp:
            for b in range(len(s.members)):
                arrays[f"y{b}"] = s.ys[b].cpu().numpy()
                arrays[f"dw{b}"] = s.dws[b].cpu().numpy()
                arrays[f"db{b}"] = s.dbs[b].cpu().numpy()
        else:
            arrays["y"] = s.y.cpu().numpy()
            arrays["dw"] = s.dw.cpu().numpy()
            arrays["db"] = s.db.cpu().numpy()
        if s.dx is not None:
            arrays["dx"] = s.dx.cpu().numpy()
        for k, v in arrays.items():
            np.save(os.path.join(path, f"u{i}_{k}.npy"), v)
        u["arrays"] = sorted(arrays)
        meta["units"].append(u)
    json.dump(meta, open(os.path.join(path, "meta.json"), "w"), indent=1)


class GroupState:
    """Sibling layers that read one input, run as a fused group (one GEMM per pass; include/glp.h
    "fused sibling groups").  Same unit interface as LayerState."""

    def __init__(self, members, n_local, n_global, math, dev, grads, idxs):
        import torch
        import paper_conf_icpp_futhys18_b200 as glp
        self.glp = glp
        self.members = members
        l0 = members[0]
        self.layer = l0
        self.name = "+".join(m.name for m in members)
        self.n = n_local
        self.conv = glp.ConvLayer(n_local, l0.C, l0.H, l0.W, None, l0.K, l0.S, l0.P, math=math,
                                  device=dev.index, branches=[m.Co for m in members],
                                  options=PLAN_OPTIONS or None)
        ds = [gen_layer(m, n_global=n_global, batch=n_local) for m in members]
        self.host = {"x": torch.from_numpy(ds[0]["x"])}   # the shared input
        for i, d in enumerate(ds):
            for k in ("w", "b", "dy"):
                self.host[f"{k}{i}"] = torch.from_numpy(d[k])
        self.t = {k: v.to(dev) for k, v in self.host.items()}
        nb = len(members)
        self.ws = [self.t[f"w{i}"] for i in range(nb)]
        self.bs = [self.t[f"b{i}"] for i in range(nb)]
        self.dys = [self.t[f"dy{i}"] for i in range(nb)]
        self.ys = [torch.empty(s, device=dev) for s in self.conv.branch_y_shapes()]
        self.dx = None if l0.data_fed else torch.empty(self.conv.x_shape, device=dev)
        self.dws = [grads.dw(i) for i in idxs]
        self.dbs = [grads.db(i) for i in idxs]
        self.flops = float(sum(m.with_batch(n_local).flops_per_pass() for m in members))
        self.idxs = list(idxs)
        self.owner, self.has_sharer, self.accumulate, self.shared_keys = None, False, False, set()

    def grad_idxs(self):
        return self.idxs

    def launches(self):
        nb = len(self.members)   # per-branch packs of W (x2) and dy
        return 6 + 3 * nb if self.dx is not None else 5 + 2 * nb

    def pack_x(self, st=None):
        self.conv.stage_pack_group(self.glp.GLP_PACK_X, [self.t["x"]], stream=st)

    def pack_w_fwd(self, st=None):
        self.conv.stage_pack_group(self.glp.GLP_PACK_W_FWD, self.ws, stream=st)

    def fwd(self, st=None):
        self.conv.stage_fwd_group(self.bs, self.ys, stream=st)

    def pack_dy(self, st=None):
        self.conv.stage_pack_group(self.glp.GLP_PACK_DY_DB, self.dys, stream=st)

    def pack_w_bwd(self, st=None):
        self.conv.stage_pack_group(self.glp.GLP_PACK_W_BWD_DATA, self.ws, stream=st)

    def bwd_data(self, st=None):
        self.conv.stage_bwd_data(self.dx, stream=st)

    def bwd_filter(self, st=None):
        self.conv.stage_bwd_filter(stream=st)

    def reduce(self, st=None):
        self.conv.stage_reduce_group(self.dws, self.dbs, stream=st)


def run_pool(args):
    """The paper's stream-pool scheme (include/glp.h glp_pool_*) on the same workload: every
    layer-pass as per-sample kernels over a pool of streams.  Comparator only (1 GPU, eager)."""
    import torch
    import paper_conf_icpp_futhys18_b200 as glp
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    layers = config(args.workload)
    units = []
    for l in layers:
        d = gen_layer(l)
        t = {k: torch.from_numpy(v).to(dev) for k, v in d.items()}
        pool = glp.StreamPool(l.N, l.C, l.H, l.W, l.Co, l.K, l.S, l.P, math=args.math,
                              n_streams=args.pool_streams)
        y = torch.empty(l.y_shape, device=dev)
        # "profile once" (P173): the CUPTI resource tracker measures T_K and T_launch in one run,
        # and Eq. 7's launch term resizes the pool
        pool.fwd(t["x"], t["w"], t["b"], y)
        pool.calibrate(t["x"], t["w"], t["b"], y)
        dx = None if l.data_fed else torch.empty(l.x_shape, device=dev)
        dw = torch.empty(l.w_shape, device=dev)
        db = torch.empty(l.Co, device=dev)
        units.append((l, pool, t, y, dx, dw, db))

    def step():
        for l, pool, t, y, dx, dw, db in units:
            pool.fwd(t["x"], t["w"], t["b"], y)
        for l, pool, t, y, dx, dw, db in reversed(units):
            pool.bwd(t["x"], t["dy"], t["w"], dx, dw, db)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    def timed(fn):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.steps):
            fn()
        e1.record()
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / args.steps

    ms_eager = timed(step)
    # the same per-sample launches recorded once into a CUDA graph (the pool's fork/join events
    # are captured as graph edges), removing the host launch cost the eager pool pays
    ms_graph = None
    if not args.no_graph:
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            step()
        g.replay()
        torch.cuda.synchronize()
        ms_graph = timed(g.replay)
    ms = min(ms_eager, ms_graph or ms_eager)
    step_flops = sum(l.flops_per_pass() * (2 if l.data_fed else 3) for l in layers)
    print(json.dumps({
        "metric": METRIC, "value": round(layers[0].N / (ms / 1e3), 1), "unit": UNIT, "n_gpus": 1,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 4),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": DTYPE[args.math],
        "data": "synthetic (seeded, Table 5 shapes; glp_workloads)",
        "scheme": "stream-pool (paper's prior-art scheme: per-sample kernels, round-robin streams)",
        "config": {"workload": CONFIG_NAMES[args.workload], "model": "conv layers only",
                   "global_batch": layers[0].N, "layers": [l.name for l in layers],
                   "pool_streams": [u[1].n_streams for u in units],
                   "eq7_bound": [u[1].eq7_bound for u in units],
                   "eq7_launch_bound": [u[1].eq7_launch_bound for u in units],
                   "t_kernel_us": [round(u[1].t_kernel_us, 2) for u in units],
                   "t_launch_us": [round(u[1].t_launch_us, 2) for u in units]},
        "launch": "cuda_graph" if ms_graph is not None and ms_graph <= ms_eager else "eager",
        "ms_per_step_eager": round(ms_eager, 4),
        "ms_per_step_graph": None if ms_graph is None else round(ms_graph, 4),
        "tflops_step": round(step_flops / (ms * 1e-3) / 1e12, 1)}), flush=True)


def build_states(args, math, G, rank, dev, grads, leaves=0):
    """Plans, seeded inputs and outputs of every unit of the workload at this rank's batch."""
    from paper_conf_icpp_futhys18_b200.dist import shard_range
    layers = config(args.workload)
    shards = [shard_range(l.N, rank, G) for l in layers]
    if args.scaling == "strong":
        n_local = [b - a for a, b in shards]
        n_global = [l.N for l in layers]
    else:
        n_local = [l.N for l in layers]
        n_global = [l.N * G for l in layers]
    groups = [] if args.no_fuse else SIBLINGS.get(args.workload, [])
    in_group = {name: gi for gi, g in enumerate(groups) for name in g}
    states = []
    done_groups = set()
    for i, (l, nl, ng) in enumerate(zip(layers, n_local, n_global)):
        shard = shards[i] if args.scaling == "strong" and G > 1 else None
        gi = in_group.get(l.name)
        if gi is None:
            states.append(LayerState(l, nl, ng, shard, math, dev, grads, i, leaves))
        elif gi not in done_groups:
            if shard is not None:
                raise SystemExit("fused groups with strong scaling: use --no-fuse")
            done_groups.add(gi)
            idxs = [j for j, m in enumerate(layers) if m.name in groups[gi]]
            states.append(GroupState([layers[j] for j in idxs], nl, ng, math, dev, grads, idxs))
    by_name = {s.name: s for s in states}
    for sharer, owner in SHARED.get(args.workload, {}).items():
        by_name[sharer].share_params_of(by_name[owner])
    return layers, states, n_local


def dag_levels(args, states):
    """Network DAG levels of the workload's units (glp_workloads.LEVELS; default: a chain)."""
    lv = None if args.chain else LEVELS.get(args.workload)
    if not lv:
        return [[i] for i in range(len(states))]
    where = {name: k for k, names in enumerate(lv) for name in names}
    unit_level = [where[(s.members[0] if isinstance(s, GroupState) else s.layer).name]
                  for s in states]
    levels = [[i for i, u in enumerate(unit_level) if u == k] for k in range(len(lv))]
    # within a level, parameter owners are issued before their sharers (the sharer's accumulate=1
    # reduction waits for the owner's)
    levels = [sorted(l, key=lambda i: states[i].owner is not None) for l in levels]
    return [l for l in levels if l]


class Step:
    """One training step of every unit's hot path, issued as the stream DAG of a real network's
    step (or serially, with CUDA events around each GEMM, for the per-kernel attribution).

    Gradient exchange (G > 1, BJ.ns (4)): 'nccl' = every unit's dW||db bucket is
    all-reduced (SUM, NCCL over NVLink) on its filter-gradient stream as soon as that unit's
    filter-gradient GEMM and reductions are done -- in reverse layer order, overlapping the
    remaining backward-data work of the earlier layers; the step ends when every bucket has
    arrived.  'tree' = the deterministic exchange (NEXT-2) after the step."""

    def __init__(self, args, states, grads, G, dev, tree=None):
        import torch
        self.args, self.states, self.grads, self.G = args, states, grads, G
        self.tree = tree
        self.levels = dag_levels(args, states)
        self.width = max(len(l) for l in self.levels)
        self.side_w = torch.cuda.Stream(device=dev)   # weight packs (known at step start)
        self.fstreams = [None] + [torch.cuda.Stream(device=dev) for _ in range(self.width - 1)]
        self.gstreams = [torch.cuda.Stream(device=dev) for _ in range(self.width)]
        self.bucketed = G > 1 and tree is None
        self.works = []

    def _bucket(self, s, g):
        """All-reduce this unit's gradient bucket(s) on stream g (after its reductions); a parameter
        owner with a sharer leaves its bucket to the sharer (issued after the accumulation)."""
        if not self.bucketed or s.has_sharer:
            return
        import torch
        import torch.distributed as dist
        with torch.cuda.stream(g):
            self.works.append(dist.all_reduce(self.grads.bucket(s.grad_idxs()),
                                              op=dist.ReduceOp.SUM, async_op=True))

    def exchange_tail(self):
        """Join the exchange: bucketed all-reduces (already in flight) or the tree."""
        if self.tree is not None:
            self.tree(self.grads.buf)
        for w in self.works:
            w.wait()   # the current stream waits for the collective
        self.works = []

    def __call__(self, ev=None, concurrent=None, with_exchange=True):
        import torch
        states = self.states
        stream = torch.cuda.current_stream()   # the capture stream while a graph is recorded
        conc = (ev is None) if concurrent is None else concurrent

        def mark(e):
            # attribution runs: a GPU-side spin before each start event keeps the stream busy while
            # the host enqueues the event and the kernel, so the interval holds the kernel only
            torch.cuda._sleep(40000)
            e.record(stream)

        if not conc:
            for i, s in enumerate(states):
                s.pack_x()
                s.pack_w_fwd()
                if ev is not None:
                    mark(ev[i][0])
                s.fwd()
                if ev is not None:
                    ev[i][1].record(stream)
            for i in reversed(range(len(states))):
                s = states[i]
                s.pack_dy()
                if s.dx is not None:
                    s.pack_w_bwd()
                    if ev is not None:
                        mark(ev[i][2])
                    s.bwd_data()
                    if ev is not None:
                        ev[i][3].record(stream)
                if ev is not None:
                    mark(ev[i][4])
                s.bwd_filter()
                if ev is not None:
                    ev[i][5].record(stream)
                s.reduce()
                if with_exchange:
                    self._bucket(s, stream)
            if with_exchange:
                self.exchange_tail()
            return
        fs = [stream] + self.fstreams[1:]
        side_w, gstreams = self.side_w, self.gstreams
        side_w.wait_stream(stream)
        for g in gstreams:
            g.wait_stream(stream)
        ew_f, ew_b, red_done = {}, {}, {}
        with torch.cuda.stream(side_w):
            for i, s in enumerate(states):
                s.pack_w_fwd(side_w)
                ew_f[i] = torch.cuda.Event()
                ew_f[i].record(side_w)
            for i in reversed(range(len(states))):
                s = states[i]
                if s.dx is not None:
                    s.pack_w_bwd(side_w)
                ew_b[i] = torch.cuda.Event()
                ew_b[i].record(side_w)

        def fork(n):
            for k in range(1, n):
                fs[k].wait_stream(stream)

        def join(n):
            for k in range(1, n):
                stream.wait_stream(fs[k])

        for lvl in self.levels:
            fork(len(lvl))
            for k, i in enumerate(lvl):
                s, f = states[i], fs[k]
                with torch.cuda.stream(f):
                    s.pack_x(f)
                    f.wait_event(ew_f[i])
                    s.fwd(f)
            join(len(lvl))
        for lvl in reversed(self.levels):
            fork(len(lvl))
            for k, i in enumerate(lvl):
                s, f, g = states[i], fs[k], gstreams[k]
                with torch.cuda.stream(f):
                    s.pack_dy(f)
                    e_dy = torch.cuda.Event()
                    e_dy.record(f)
                    g.wait_event(e_dy)
                    with torch.cuda.stream(g):
                        s.bwd_filter(g)
                        if s.owner is not None:   # accumulate onto the owner's finished gradient
                            g.wait_event(red_done[id(s.owner)])
                        s.reduce(g)
                        red_done[id(s)] = torch.cuda.Event()
                        red_done[id(s)].record(g)
                    if with_exchange:
                        self._bucket(s, g)
                    if s.dx is not None:
                        f.wait_event(ew_b[i])
                        s.bwd_data(f)
            join(len(lvl))
        stream.wait_stream(side_w)
        for g in gstreams:
            stream.wait_stream(g)
        if with_exchange:
            self.exchange_tail()


def time_steps(step_fn, steps, stream):
    """Device time of `steps` calls of step_fn (CUDA events on `stream`), ms per step."""
    import torch
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    t0.record(stream)
    for _ in range(steps):
        step_fn()
    t1.record(stream)
    torch.cuda.synchronize()
    return t0.elapsed_time(t1) / steps


def quick_mode(args, math, G, rank, dev):
    """Images/s of the same workload in another math mode (1 GPU, CUDA-graph replay): the
    bf16 / tf32 lines reported beside the fp32 headline."""
    import torch
    from paper_conf_icpp_futhys18_b200.dist import FlatGrads
    layers = config(args.workload)
    grads = FlatGrads([l.w_shape for l in layers], device=dev)
    _, states, n_local = build_states(args, math, G, rank, dev, grads)
    step = Step(args, states, grads, G, dev)
    for _ in range(max(3, args.warmup)):
        step()
    g_step = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g_step):
        step(concurrent=not args.serial, with_exchange=False)
    for _ in range(3):
        g_step.replay()
    ms = time_steps(g_step.replay, args.steps, torch.cuda.current_stream())
    out = {"value": round(n_local[0] / (ms / 1e3), 1), "ms_per_step": round(ms, 4),
           "dtype": math, "launch": "cuda_graph"}
    del g_step, step, states
    torch.cuda.empty_cache()
    return out


def weak_scaling(args, G, rank, dev):
    """G > 1: the same step with the config batch on EVERY rank (weak scaling), reported beside the
    strong-scaling headline; eager steps with the bucketed exchange, max over ranks."""
    import argparse as _ap
    import torch
    import torch.distributed as dist
    from paper_conf_icpp_futhys18_b200.dist import FlatGrads
    a = _ap.Namespace(**vars(args))
    a.scaling = "weak"
    layers = config(a.workload)
    grads = FlatGrads([l.w_shape for l in layers], device=dev)
    _, states, n_local = build_states(a, a.math, G, rank, dev, grads)
    step = Step(a, states, grads, G, dev)
    for _ in range(max(3, a.warmup)):
        step()
    torch.cuda.synchronize()
    dist.barrier()
    ms = time_steps(lambda: step(concurrent=not a.serial), a.steps, torch.cuda.current_stream())
    tt = torch.tensor([ms], device=dev)
    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    ms = float(tt.item())
    out = {"value": round(n_local[0] * G / (ms / 1e3), 1), "ms_per_step": round(ms, 4),
           "per_gpu_batch": n_local[0], "global_batch": n_local[0] * G}
    del step, states
    torch.cuda.empty_cache()
    return out


def run_glp(args, ws, rank, local):
    import torch
    import torch.distributed as dist

    dev = torch.device("cuda", 0 if args.same_device else local)
    torch.cuda.set_device(dev)
    G = ws
    if G > 1:
        if args.dist_backend == "nccl":
            # the NCCL communicator lines (ring/tree/NVLS choice over NVLink) go to stderr
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")
    from paper_conf_icpp_futhys18_b200.dist import FlatGrads
    layers = config(args.workload)
    grads = FlatGrads([l.w_shape for l in layers], device=dev)
    flat = grads.buf
    nparams = grads.numel
    tree, n_leaves = None, 0
    if args.exchange == "tree":
        from paper_conf_icpp_futhys18_b200.dist import LeafTreeExchange, rank_leaves
        n_leaves = len(rank_leaves(rank, G))
        if SIBLINGS.get(args.workload) and not args.no_fuse:
            raise SystemExit("--exchange tree: single layers only (use --no-fuse)")
        if SHARED.get(args.workload):
            raise SystemExit("--exchange tree: no shared-parameter workloads")
    layers, states, n_local = build_states(args, args.math, G, rank, dev, grads, n_leaves)
    if args.exact_data:
        set_exact_data(states)
    stream = torch.cuda.current_stream()
    if args.exchange == "tree":
        # the step packs once; each unit's filter gradient reduces per leaf into the exchange's leaf
        # buffers; the fixed 8-leaf tree (local subtree + top levels across ranks) gives dW||db
        tree = LeafTreeExchange(grads.numel, n_leaves, dev)
        for s in states:
            s.leaves, s.slot = tree, grads.slots[s.idx]
    step = Step(args, states, grads, G, dev, tree)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if G > 1:
        dist.barrier()
    # One GPU: the whole step (every pack, GEMM and reduction launch of all layers) is recorded
    # once as a CUDA graph and replayed.  G > 1: the step is issued eagerly so that each unit's
    # gradient bucket is all-reduced (NCCL) as soon as it is ready, overlapping the rest of the
    # backward (NCCL collectives are not captured into the graph).
    use_graph = not args.no_graph and G == 1
    evs = [[[torch.cuda.Event(enable_timing=True) for _ in range(6)] for _ in states]
           for _ in range(args.steps)]
    if use_graph:
        g_step = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g_step):
            step(concurrent=not args.serial, with_exchange=False)
        for _ in range(max(1, args.warmup)):
            g_step.replay()
            step.exchange_tail()

        def run_one():
            g_step.replay()
            step.exchange_tail()   # the tree kernel (tree mode); nothing on one GPU otherwise
    else:
        def run_one():
            step(concurrent=not args.serial)
    clocks = ClockSampler(dev.index) if rank == 0 else None
    if clocks:
        clocks.start()
    if G > 1:
        torch.cuda.synchronize()
        dist.barrier()
    ms_per_step = time_steps(run_one, args.steps, stream)
    if G > 1:
        dist.barrier()
    clk = clocks.stop() if clocks else None
    if G > 1:
        tt = torch.tensor([ms_per_step], device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_per_step = float(tt.item())
    images_per_step = sum(n_local[:1]) * G if args.scaling == "weak" else layers[0].N
    value = images_per_step / (ms_per_step / 1e3)

    # per-kernel attribution: events cannot time nodes inside a graph, so the same step runs K
    # more times eagerly and serially with CUDA events around each GEMM on the launching stream
    # (kernel durations do not depend on how the launches were issued)
    for k in range(args.steps):
        step(evs[k], concurrent=False, with_exchange=False)
    torch.cuda.synchronize()
    kern = []
    for i, s in enumerate(states):
        for name, a, b in (("fwd", 0, 1), ("bwd_data", 2, 3), ("bwd_filter", 4, 5)):
            if name == "bwd_data" and s.dx is None:
                continue
            us = [evs[k][i][a].elapsed_time(evs[k][i][b]) * 1e3 for k in range(args.steps)]
            avg = sum(us) / len(us)
            kern.append({"layer": s.name, "pass": name, "avg_us": round(avg, 2),
                         "total_us": sum(us), "tflops": round(s.flops / (avg * 1e-6) / 1e12, 1)})
    if args.dump:
        # one more full step (with the exchange): the attribution steps above skip it, so dW || db
        # would hold this rank's unreduced gradients
        step()
        torch.cuda.synchronize()
        if rank == 0:
            dump_units(states, args.dump, args.workload, args.math)
    roofline = make_roofline(args, states, kern, ms_per_step)
    step_flops = sum(s.flops * (3 if s.dx is not None else 2) for s in states)

    # end-to-end through the public API: pinned host buffers -> device every step (each unit's
    # x, dy, W, b), the step, and dW||db back to the host every step
    e2e = None
    if not args.no_e2e:
        host_pinned = [{k: v.pin_memory() for k, v in s.host.items() if k not in s.shared_keys}
                       for s in states]
        out_host = torch.empty(nparams, pin_memory=True)
        h2d_bytes = sum(v.numel() * 4 for hp in host_pinned for v in hp.values())
        d2h = nparams * 4
        ke = max(1, args.e2e_steps)
        step()
        torch.cuda.synchronize()
        if G > 1:
            dist.barrier()

        # Pipelined like a training input loader: step k+1's inputs travel host -> device (a
        # copy stream, into device staging buffers) while step k computes; each step starts with
        # a device-to-device copy staging -> the step's own input tensors (the captured graph's
        # addresses).  The timed region holds all K host -> device copies (the first one not
        # overlapped), K steps and K device -> host reads of dW||db.
        staging = [{k2: torch.empty_like(s.t[k2]) for k2 in hp} for s, hp in zip(states, host_pinned)]
        cs = torch.cuda.Stream(device=dev)

        def h2d():
            with torch.cuda.stream(cs):
                for st_, hp in zip(staging, host_pinned):
                    for k2, v in hp.items():
                        st_[k2].copy_(v, non_blocking=True)
            ev = torch.cuda.Event()
            ev.record(cs)
            return ev

        def e2e_run(k_steps):
            ready = h2d()
            for k in range(k_steps):
                stream.wait_event(ready)
                for s, st_ in zip(states, staging):
                    for k2, v in st_.items():
                        s.t[k2].copy_(v, non_blocking=True)
                if k + 1 < k_steps:
                    consumed = torch.cuda.Event()
                    consumed.record(stream)
                    cs.wait_event(consumed)
                    ready = h2d()
                step()
                out_host.copy_(flat, non_blocking=True)

        e2e_run(1)   # warm the copy path
        torch.cuda.synchronize()
        ems = time_steps(lambda: e2e_run(ke), 1, stream) / ke
        if G > 1:
            tt = torch.tensor([ems], device=dev)
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            ems = float(tt.item())
        e2e = {"value": round(images_per_step / (ems / 1e3), 1), "unit": UNIT,
               "h2d_bytes_per_step": int(h2d_bytes), "d2h_bytes_per_step": int(d2h),
               "ms_per_step": round(ems, 3), "steps": ke,
               "pipelined": "step k+1's host->device copy overlaps step k (copy stream + device staging)"}

    weak = None
    if G > 1 and args.scaling == "strong" and not args.no_extra_modes:
        weak = weak_scaling(args, G, rank, dev)
    modes = None
    if G == 1 and not args.no_extra_modes:
        modes = {m: quick_mode(args, m, G, rank, dev) for m in ("bf16", "tf32") if m != args.math}

    # kernels per timed step, counted (not modelled): the CUPTI tracker (libglp_tracker.so, the
    # NEXT-4 resource tracker) records every kernel of one more step issued exactly as the timed
    # ones; ours are the glp:: kernels.  Formula fallback where CUPTI is unavailable.
    launches_src = "formula (packs, GEMMs, reductions per unit)"
    per_step = sum(s.launches() for s in states)
    if G == 1:   # (G > 1: the step holds collectives every rank must join)
        try:
            from paper_conf_icpp_futhys18_b200.tracker import Tracker
            torch.cuda.synchronize()
            with Tracker() as trk:
                run_one()
                torch.cuda.synchronize()
            ours = [k for k in trk.kernels if "glp" in k.name]
            if ours:
                per_step = len(ours)
                launches_src = (f"CUPTI kernel records of one extra step issued like the timed ones "
                                f"({len(ours)} glp kernels, {len(trk.kernels) - len(ours)} other)")
        except Exception as e:   # no CUPTI / tracker library: keep the formula
            launches_src += f"; tracker unavailable: {type(e).__name__}"

    cpu = None
    if rank == 0 and G == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(layers, budget_s=12.0)

    if G > 1:
        dist.barrier()
    if rank != 0:
        if G > 1:
            dist.destroy_process_group()
        return
    info0 = [s.conv.info for s in states]
    knobs = {k: v for k, v in os.environ.items() if k.startswith("GLP_")}
    line = {
        "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": G,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 4),
        "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None,
        "dtype": DTYPE[args.math], "data": "synthetic (seeded, Table 5 shapes; glp_workloads)",
        "config": {"workload": CONFIG_NAMES[args.workload], "model": "conv layers only",
                   "global_batch": images_per_step, "per_gpu_batch": n_local[0],
                   "layers": [s.name for s in states], "math": args.math,
                   "parallelism": f"dp{G}", "exchange": args.exchange + (
                       " (per-unit buckets overlapped with the backward)" if step.bucketed else ""),
                   "l2": "inputs larger than L2 (step working set "
                   f"{sum(v.numel() * 4 for s in states for v in s.t.values()) / 1e9:.2f} GB)",
                   "step_gflop": round(step_flops / 1e9, 1),
                   "samples_in_flight": [i.samples_in_flight for i in info0],
                   "wgrad_splits": [i.splits_wgrad for i in info0],
                   **({"plan_options": PLAN_OPTIONS} if PLAN_OPTIONS else {})},
        "tflops_step": round(step_flops / (ms_per_step * 1e-3) / 1e12, 1),
        "roofline": roofline,
        "kernels": [{k: r[k] for k in ("layer", "pass", "avg_us", "tflops")} for r in kern],
        "modes": modes,
        "weak_scaling": weak,
        "cpu_baseline": cpu,
        "clocks": clk,
        "e2e": e2e,
        "gpu_launches": int(per_step * args.steps),
        "gpu_launches_source": launches_src,
        "launch": ("cuda_graph" if use_graph else "eager") +
                  ("" if args.serial else
                   f" (step DAG: {len(step.levels)} levels, up to {step.width} concurrent units)"),
        "env_knobs": knobs,
    }
    print(json.dumps(line), flush=True)
    if G > 1:
        dist.destroy_process_group()


def make_roofline(args, states, kern, ms_per_step):
    """Roofline of the dominant kernel (largest share of the step): achieved = its algorithmic
    flops per launch / its live CUDA-event duration; peak = the measured burst bf16 figure of
    MEASURED_PEAKS.json (the kernel is event-timed alone, in a sub-second region) times the
    guide's nominal ratio for the kernel's dtype (tf32: 1.1/2.25; 3xTF32: three tf32 MMAs per
    fp32-equivalent flop, /3).  The sustained figure is given as context."""
    peaks = load_peaks()
    dom = max(kern, key=lambda r: r["total_us"])
    # fp32: the dominant kernel's own split -- 3xTF32 (three tf32 MMAs per flop: tf32 peak / 3)
    # or the mixed split (one tf32 + two bf16 MMAs, bf16 at twice the tf32 rate: tf32 peak / 2)
    mixed = args.math == "fp32" and any(getattr(s.conv.info, "fp32_split", 0) for s in states
                                        if dom["layer"] == s.name)
    ratio = {"bf16": 1.0, "tf32": NOMINAL_TF32_OVER_BF16,
             "fp32": NOMINAL_TF32_OVER_BF16 / (2 if mixed else 3)}[args.math]
    peak_tf = peaks["bf16_tflops"] * ratio
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        try:
            traffic = json.load(open(tpath)).get(f"{args.workload}/{dom['layer']}/{dom['pass']}/{args.math}")
        except Exception:
            traffic = None
    src = {"bf16": " bf16 burst", "tf32": " bf16 burst x 1.1/2.25 (tf32)",
           "fp32": (" bf16 burst x 1.1/2.25 / 2 (mixed split: one tf32 + two bf16 MMAs per flop)"
                    if mixed else " bf16 burst x 1.1/2.25 / 3 (3xTF32: three tf32 MMAs per flop)")}[args.math]
    out = {"bound": "tensor", "achieved": dom["tflops"], "peak": round(peak_tf, 1),
           "unit": "TFLOP/s", "frac": round(dom["tflops"] / peak_tf, 4), "traffic": traffic,
           "kernel": f"{kernel_name(states, dom)} {dom['layer']} {dom['pass']}",
           "peak_source": peaks["source"] + src,
           "share_of_step": round(dom["total_us"] / 1e3 / (ms_per_step * args.steps), 4),
           "frac_of_sustained_peak": round(dom["tflops"] / (peaks["bf16_tflops_sustained"] * ratio), 4)}
    if args.math == "fp32":
        # the same kernel against the tensor pipe's nominal tf32 rate (1.1 PF/s dense, /2 or /3)
        out["frac_of_nominal_tf32"] = round(dom["tflops"] / (1100.0 / (2 if mixed else 3)), 4)
        out["fp32_split"] = "tf32 hi*hi + 2 bf16 cross terms" if mixed else "3xTF32"
    return out


# ------------------------------------------------------------------------- CPU oracle --------

def _oracle_items(layers, n):
    items = []
    for l in layers:
        lb = l.with_batch(n)
        f = lb.flops_per_pass()
        items.append((l, "fwd", f))
        items.append((l, "bwd_filter", f))
        if not l.data_fed:
            items.append((l, "bwd_data", f))
    return items


def _oracle_run(l, kind, d):
    import oracle
    G = l.groups   # grouped layers: one oracle convolution per group (independent convolutions)
    cg, og = l.C // G, l.Co // G
    for g in range(G):
        x = d["x"][:, g * cg:(g + 1) * cg]
        w = d["w"][g * og:(g + 1) * og]
        dy = d["dy"][:, g * og:(g + 1) * og]
        if kind == "fwd":
            oracle.conv_fwd(x, w, d["b"][g * og:(g + 1) * og], l.S, l.P)
        elif kind == "bwd_filter":
            oracle.conv_bwd_filter(x, dy, w.shape, l.S, l.P)
        else:
            oracle.conv_bwd_data(dy, w, x.shape, l.S, l.P)


def cpu_baseline(layers, budget_s=12.0, n_sample=None):
    """The fp64 oracle (as it stands) on a bounded sample: batches of `n` images through every
    layer-pass of the step until the time budget is used; images/s = images done / time."""
    import oracle
    cores = oracle.max_threads()
    n = n_sample or max(1, min(layers[0].N, cores))
    data = {l.name: gen_layer(l, batch=n) for l in layers}
    items = _oracle_items(layers, n)
    done_flops, t_used = 0.0, 0.0
    per_image = sum(f for _, _, f in items) / n
    passes = 0
    while True:
        for l, kind, f in items:
            t0 = time.perf_counter()
            _oracle_run(l, kind, data[l.name])
            t_used += time.perf_counter() - t0
            done_flops += f
            if t_used >= budget_s:
                break
        passes += 1
        if t_used >= budget_s:
            break
    images = done_flops / per_image
    return {"value": round(images / t_used, 4), "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{images:.3f} images (batches of {n}, every layer-pass of the step, "
                      f"{t_used:.1f} s, fp64 direct loops, OpenMP)"}


def run_reference(args, ws, rank):
    if rank != 0:
        return
    import oracle
    layers = config(args.workload)
    cores = oracle.max_threads()
    total = args.steps + args.warmup
    budget_total = 150.0
    per_step = min(5.0, max(0.5, budget_total / max(1, total)))
    n = max(1, min(layers[0].N, cores))
    data = {l.name: gen_layer(l, batch=n) for l in layers}
    items = _oracle_items(layers, n)
    per_image = sum(f for _, _, f in items) / n
    it = 0
    times, flops = [], []

    def one_step():
        nonlocal it
        t_used, f_done = 0.0, 0.0
        while t_used < per_step:
            l, kind, f = items[it % len(items)]
            it += 1
            t0 = time.perf_counter()
            _oracle_run(l, kind, data[l.name])
            t_used += time.perf_counter() - t0
            f_done += f
        return t_used, f_done

    for _ in range(args.warmup):
        one_step()
    for _ in range(args.steps):
        t, f = one_step()
        times.append(t)
        flops.append(f)
    images = sum(flops) / per_image
    value = images / sum(times)
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": UNIT,
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(sum(times) / len(times) * 1e3, 2), "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
        "data": "synthetic (seeded, Table 5 shapes; glp_workloads)",
        "config": {"workload": CONFIG_NAMES[args.workload], "model": "conv layers only",
                   "global_batch": layers[0].N, "layers": [l.name for l in layers]},
        "cpu_baseline": {"value": round(value, 4), "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": f"each step = {per_step:.1f} s of oracle layer-passes on a "
                                   f"{n}-image batch; {images:.3f} images total"},
        "e2e": {"value": round(value, 4), "unit": UNIT, "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def free_port() -> int:
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def relaunch(args) -> int:
    """`python bench.py --gpus N` (N > 1) outside torchrun: start the N ranks ourselves (one
    process per GPU) with torch.distributed.run on 127.0.0.1; rank 0 prints the line."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr", "127.0.0.1",
           "--master-port", str(free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def dry_run(ws, rank):
    """Launcher plumbing check on CPU (gloo): every rank contributes 1, rank 0 prints the count."""
    import torch
    import torch.distributed as dist
    if ws > 1:
        dist.init_process_group("gloo")
    t = torch.ones(1)
    if ws > 1:
        dist.all_reduce(t)
    if rank == 0:
        print(json.dumps({"metric": METRIC, "n_gpus": ws, "ranks_seen": int(t.item()),
                          "dry_run": True}), flush=True)
    if ws > 1:
        dist.destroy_process_group()


def main():
    args = parse_args()
    ws, rank, local = dist_env()
    if args.impl == "reference":
        run_reference(args, ws, rank)
        return
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        sys.exit(relaunch(args))
    if ws != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws}: refusing to run a different "
                 "number of ranks than asked")
    diag = sorted(k for k in os.environ if k.startswith("GLP_DEBUG"))
    if diag:
        sys.exit(f"bench.py: diagnostic knob(s) {diag} set: they skip work in -DGLP_DIAG builds, so "
                 "no throughput is printed (unset them)")
    if args.dry_run:
        dry_run(ws, rank)
        return
    import torch
    if torch.cuda.device_count() < (1 if args.same_device else local + 1):
        sys.exit(f"bench.py: rank {rank} needs cuda:{local} but {torch.cuda.device_count()} "
                 "CUDA device(s) are visible (there is no CPU fallback)")
    if args.plan_options:
        PLAN_OPTIONS.update(json.loads(args.plan_options))
    if args.scheme == "pool":
        if rank == 0:
            run_pool(args)
        return
    run_glp(args, ws, rank, local)


if __name__ == "__main__":
    main()
