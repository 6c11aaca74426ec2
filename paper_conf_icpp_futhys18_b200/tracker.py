"""Python binding of libglp_tracker.so (include/glp_tracker.h): the paper's CUPTI resource
tracker (§3.1 P165, "profile once, execute many" P173).

Argument marshalling only.  ``Tracker`` collects, between start() and stop(), every kernel the
process ran (name, grid, block, cluster, registers, shared memory, timestamps) and every
kernel-launch API call; the stream-pool comparator turns them into Eq. 7's T_K / T_launch.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import List

PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(PKG, "libglp_tracker.so")
_lib = None


class KernelRecord(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 128), ("grid", ctypes.c_int * 3), ("block", ctypes.c_int * 3),
                ("cluster", ctypes.c_int * 3), ("regs", ctypes.c_int), ("static_smem", ctypes.c_int),
                ("dynamic_smem", ctypes.c_int), ("queued_ns", ctypes.c_uint64),
                ("submitted_ns", ctypes.c_uint64), ("start_ns", ctypes.c_uint64),
                ("end_ns", ctypes.c_uint64), ("stream_id", ctypes.c_uint32),
                ("correlation_id", ctypes.c_uint32)]


class LaunchRecord(ctypes.Structure):
    _fields_ = [("start_ns", ctypes.c_uint64), ("end_ns", ctypes.c_uint64),
                ("correlation_id", ctypes.c_uint32), ("driver", ctypes.c_int)]


EXPORTS = ["glp_tracker_start", "glp_tracker_stop", "glp_tracker_clear", "glp_tracker_kernel_count",
           "glp_tracker_kernel", "glp_tracker_launch_count", "glp_tracker_launch",
           "glp_tracker_last_error"]


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        L.glp_tracker_kernel.argtypes = [ctypes.c_int, ctypes.POINTER(KernelRecord)]
        L.glp_tracker_launch.argtypes = [ctypes.c_int, ctypes.POINTER(LaunchRecord)]
        L.glp_tracker_last_error.restype = ctypes.c_char_p
        _lib = L
    return _lib


@dataclass
class Kernel:
    name: str
    grid: tuple
    block: tuple
    cluster: tuple
    regs: int
    smem: int
    start_ns: int
    end_ns: int
    submitted_ns: int

    @property
    def duration_us(self) -> float:
        return (self.end_ns - self.start_ns) / 1e3


class Tracker:
    """Context manager: `with Tracker() as t: ...` then t.kernels / t.launch_us."""

    def __init__(self):
        self.kernels: List[Kernel] = []
        self.launch_us: List[float] = []

    def start(self):
        L = lib()
        L.glp_tracker_clear()
        if L.glp_tracker_start() != 0:
            raise RuntimeError(f"glp_tracker_start: {L.glp_tracker_last_error().decode()}")
        return self

    def stop(self):
        import torch
        torch.cuda.synchronize()
        L = lib()
        if L.glp_tracker_stop() != 0:
            raise RuntimeError(f"glp_tracker_stop: {L.glp_tracker_last_error().decode()}")
        r = KernelRecord()
        for i in range(L.glp_tracker_kernel_count()):
            L.glp_tracker_kernel(i, ctypes.byref(r))
            self.kernels.append(Kernel(r.name.decode(errors="replace"), tuple(r.grid), tuple(r.block),
                                       tuple(r.cluster), r.regs, r.static_smem + r.dynamic_smem,
                                       r.start_ns, r.end_ns, r.submitted_ns))
        a = LaunchRecord()
        for i in range(L.glp_tracker_launch_count()):
            L.glp_tracker_launch(i, ctypes.byref(a))
            self.launch_us.append((a.end_ns - a.start_ns) / 1e3)
        L.glp_tracker_clear()
        return self

    def __enter__(self):
        return self.start()

    def __exit__(self, *exc):
        self.stop()
        return False
