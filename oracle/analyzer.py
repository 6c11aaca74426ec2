"""ORACLE — TEST INFRASTRUCTURE ONLY: the paper's analytical model, by enumeration.

PAPER.md §3.2 (P214-254), Eqs 1-9, and the sm_100a re-derivation of the per-kernel
blocks-per-SM term (R15/R16).  Everything here is written as brute force
(enumerate candidate integers, keep the feasible ones) so that the C++ product analyzer
(closed forms) is checked against an independent computation.

Readings: R14 objective sums over kernel instances (#K_i * tau * beta);
R15 Eq. 8 uses ceil when #beta < #SM; R17 the T_K/T_launch term of Eq. 7 is optional
(None = unbounded); R18 the stream count of a per-sample chain is the bound of the chain.
"""
from __future__ import annotations

import itertools
import math
from dataclasses import dataclass
from typing import Optional, Sequence


@dataclass
class Device:
    """Table 2 'device property' notations (P183-193)."""
    n_sm: int          # #SM
    C: int             # concurrency degree (max concurrent kernels), Eq. 6
    sm_max: int        # shared memory per SM (bytes), Eq. 4
    rho_max: int       # resident blocks per SM
    tau_max: int       # resident threads per SM, Eq. 5
    regs_max: int = 65536
    tmem_cols: int = 0  # sm_100a only


@dataclass
class Kernel:
    """Table 2 'profiling input' notations (P194-200)."""
    blocks: int        # #beta_Ki (grid size)
    threads: int       # tau_Ki
    smem: int = 0      # sm_Ki (bytes per block)
    regs: int = 0      # registers per thread
    t_kernel: Optional[float] = None   # T_Ki
    t_launch: Optional[float] = None   # T_launch
    tmem_cols: int = 0


def K40C() -> Device:
    """K40C: 15 SMs (Table 3 P290), 48 KB smem/SM (P298), Kepler C = 32 (Table 1 P56);
    2048 threads / 16 blocks per SM [ext: CUDA programming guide, CC 3.5]."""
    return Device(n_sm=15, C=32, sm_max=48 * 1024, rho_max=16, tau_max=2048)


def B200() -> Device:
    """B200 per-SM limits named by BASELINE.json north_star: 148 SMs, 64K registers,
    228 KB shared memory, 2048 threads, 32 blocks; C = 128 [ext]; TMEM 512 columns [ext]."""
    return Device(n_sm=148, C=128, sm_max=228 * 1024, rho_max=32, tau_max=2048,
                  regs_max=65536, tmem_cols=512)


def eq8_beta(k: Kernel, dev: Device, ceil: bool = True) -> int:
    """Eq. 8 (P250) blocks per SM, beta = #beta / #SM (floor in the paper; R15 ceil)."""
    return -(-k.blocks // dev.n_sm) if ceil else k.blocks // dev.n_sm


def eq7_bound(k: Kernel, dev: Device) -> int:
    """Eq. 7 (P245): #K_i <= min{ceil(T_K/T_launch), tau_max*#SM/(tau*#beta), sm_max*#SM/(sm*#beta)}.
    Integer bound = floor of the min; a missing term is unbounded."""
    terms = []
    if k.t_kernel is not None and k.t_launch:
        terms.append(math.ceil(k.t_kernel / k.t_launch))
    terms.append(dev.tau_max * dev.n_sm / (k.threads * k.blocks))
    if k.smem > 0:
        terms.append(dev.sm_max * dev.n_sm / (k.smem * k.blocks))
    return int(math.floor(min(terms)))


def milp_bruteforce(kernels: Sequence[Kernel], dev: Device, ceil_beta: bool = True):
    """Eqs 3-7 + 9 solved by exhaustive enumeration of the integer vector (#K_1..#K_N).

    maximise   tau_total = sum_i #K_i * tau_i * beta_i           (Eq. 3, reading R14)
    subject to sum_i #K_i * sm_i  * beta_i <= sm_max              (Eq. 4)
               sum_i #K_i * tau_i * beta_i <= tau_max             (Eq. 5)
               1 <= sum_i #K_i <= C                               (Eq. 6)
               #K_i <= Eq. 7 bound                                (Eq. 7)
    returns (tau_total, counts, C_out = sum #K_i)                 (Eq. 9)
    Ties are broken towards the larger C_out, then lexicographically larger counts."""
    betas = [eq8_beta(k, dev, ceil_beta) for k in kernels]
    ubs = [max(0, min(eq7_bound(k, dev), dev.C)) for k in kernels]
    best = None
    for counts in itertools.product(*[range(u + 1) for u in ubs]):
        tot = sum(counts)
        if tot < 1 or tot > dev.C:
            continue
        smem = sum(c * k.smem * b for c, k, b in zip(counts, kernels, betas))
        thr = sum(c * k.threads * b for c, k, b in zip(counts, kernels, betas))
        if smem > dev.sm_max or thr > dev.tau_max:
            continue
        key = (thr, tot, counts)
        if best is None or key > best:
            best = key
    if best is None:
        return 0, tuple(0 for _ in kernels), 0
    return best[0], best[2], best[1]


# ---------------------------- sm_100a re-derivation -------------------------------------

def regs_per_warp_alloc(regs_per_thread: int) -> int:
    """Register allocation per warp on sm_100a: 256-register units [ext: CUDA occupancy
    calculator, CC 10.0 register allocation unit size 256, warp granularity]."""
    return -(-max(regs_per_thread, 1) * 32 // 256) * 256


def ctas_per_sm_enum(threads: int, regs: int, smem: int, tmem_cols: int, dev: Device,
                     smem_reserved: int = 1024, smem_gran: int = 128) -> int:
    """Largest b in [0, rho_max] such that b CTAs fit every per-SM limit (enumeration).

    Limits: threads (Eq. 5), shared memory (Eq. 4, + 1 KB reserved per CTA [ext]),
    registers (hard on sm_100a, R16), blocks (rho_max), TMEM columns (R16)."""
    warps = -(-threads // 32)
    rpw = regs_per_warp_alloc(regs) if regs > 0 else 0
    smem_cta = -(-smem // smem_gran) * smem_gran + smem_reserved
    best = 0
    for b in range(0, dev.rho_max + 1):
        if b * warps * 32 > dev.tau_max:
            break
        if rpw and b * warps * rpw > dev.regs_max:
            break
        if b * smem_cta > dev.sm_max:
            break
        if tmem_cols and dev.tmem_cols and b * tmem_cols > dev.tmem_cols:
            break
        best = b
    return best


def samples_in_flight_enum(slots: int, tiles_per_sample: int, n_local: int) -> int:
    """S = largest s in [1, N] with s * tiles_per_sample <= slots (at least 1)."""
    s_best = 1
    for s in range(1, n_local + 1):
        if s * tiles_per_sample <= slots:
            s_best = s
    return s_best
