"""Pins for the analytical-model oracle (§3.2, Eqs 1-9)."""
import itertools

import pytest

from oracle import analyzer as A


def test_paper_worked_example_caffenet_conv1_k40c():
    """P173: im2col of CaffeNet conv1 on K40C runs as a [18,1,1] grid (512-thread blocks,
    33 regs) and the analyzer outputs 3.  Eq. 7 thread term: 2048*15/(512*18) = 3.33 -> 3;
    the smem term is unbounded (im2col uses none)."""
    k = A.Kernel(blocks=18, threads=512, smem=0, regs=33)
    assert A.eq7_bound(k, A.K40C()) == 3
    # The MILP with the per-sample chain read as one kernel (R18) reproduces C_out = 3
    # with Eq. 8 as printed (floor): beta = floor(18/15) = 1.
    tot, counts, c_out = A.milp_bruteforce([k], A.K40C(), ceil_beta=False)
    assert c_out == 3 and counts == (3,) and tot == 3 * 512


def test_same_kernel_on_b200():
    """The same kernel under the B200 limits of north_star: 2048*148/(512*18) = 32.9 -> 32."""
    k = A.Kernel(blocks=18, threads=512)
    assert A.eq7_bound(k, A.B200()) == 32


def test_eq8_floor_and_ceil():
    dev = A.B200()
    assert A.eq8_beta(A.Kernel(blocks=100, threads=128), dev, ceil=False) == 0   # R15 motivation
    assert A.eq8_beta(A.Kernel(blocks=100, threads=128), dev, ceil=True) == 1
    assert A.eq8_beta(A.Kernel(blocks=300, threads=128), dev, ceil=True) == 3


@pytest.mark.parametrize("threads,smem,blocks", [(256, 0, 40), (128, 16384, 148), (512, 4096, 30),
                                                 (64, 40000, 296)])
def test_single_kernel_milp_closed_form(threads, smem, blocks):
    """For one kernel the MILP optimum is min(Eq.7, floor(tau_max/(tau*beta)),
    floor(sm_max/(sm*beta)), C) — brute force agrees with that closed form."""
    dev = A.B200()
    k = A.Kernel(blocks=blocks, threads=threads, smem=smem)
    beta = A.eq8_beta(k, dev)
    bound = min(A.eq7_bound(k, dev), dev.tau_max // (threads * beta), dev.C)
    if smem:
        bound = min(bound, dev.sm_max // (smem * beta))
    _, counts, c_out = A.milp_bruteforce([k], dev)
    assert c_out == bound == counts[0]


def test_two_kernel_milp_is_optimal_and_feasible():
    """Two-kernel sets: the enumerated optimum satisfies Eqs 4-7 and no feasible vector beats it."""
    dev = A.Device(n_sm=4, C=8, sm_max=64 * 1024, rho_max=16, tau_max=2048)
    ka = A.Kernel(blocks=8, threads=256, smem=8192)
    kb = A.Kernel(blocks=4, threads=128, smem=16384)
    tot, counts, c_out = A.milp_bruteforce([ka, kb], dev)
    ba, bb = A.eq8_beta(ka, dev), A.eq8_beta(kb, dev)
    assert counts[0] * 256 * ba + counts[1] * 128 * bb == tot <= dev.tau_max
    assert counts[0] * 8192 * ba + counts[1] * 16384 * bb <= dev.sm_max
    assert 1 <= c_out <= dev.C
    for a, b in itertools.product(range(9), range(9)):
        if a + b < 1 or a + b > dev.C or a > A.eq7_bound(ka, dev) or b > A.eq7_bound(kb, dev):
            continue
        if a * 8192 * ba + b * 16384 * bb > dev.sm_max:
            continue
        thr = a * 256 * ba + b * 128 * bb
        if thr <= dev.tau_max:
            assert thr <= tot


def test_sm100_ctas_per_sm_enumeration():
    dev = A.B200()
    # 256 threads, 64 regs, 196 KB smem, 512 TMEM cols -> smem and TMEM both allow 1
    assert A.ctas_per_sm_enum(256, 64, 196 * 1024, 512, dev) == 1
    # TMEM limit: 256 columns -> at most 2 even if smem allowed more
    assert A.ctas_per_sm_enum(128, 32, 16 * 1024, 256, dev) == 2
    # thread limit: 1024 threads -> 2
    assert A.ctas_per_sm_enum(1024, 16, 0, 0, dev) == 2
    # register limit: 256 threads x 128 regs = 32768 regs -> 2
    assert A.ctas_per_sm_enum(256, 128, 0, 0, dev) == 2
    # block limit
    assert A.ctas_per_sm_enum(32, 16, 0, 0, dev) == 32


def test_samples_in_flight_enumeration():
    assert A.samples_in_flight_enum(148, 46, 256) == 3
    assert A.samples_in_flight_enum(148, 1, 64) == 64
    assert A.samples_in_flight_enum(148, 400, 256) == 1
