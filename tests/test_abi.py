"""CPU tests of the C ABI (no GPU): the library loads, exports every symbol include/glp.h
declares, validates arguments, refuses to run without a device (no CPU fallback), and its host
analyzer (closed forms) agrees with the oracle's enumeration of the paper's model."""
import ctypes
import os
import random
import re

import pytest

import paper_conf_icpp_futhys18_b200 as glp
from oracle import analyzer as A

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    from paper_conf_icpp_futhys18_b200 import _build
    _build.build()
    _build.build_tracker()


def header_functions(header="glp.h"):
    src = open(os.path.join(ROOT, "include", header)).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(glp_[a-z0-9_]+)\s*\(", src)))


def test_exports_every_declared_symbol():
    decl = header_functions()
    assert len(decl) >= 15
    assert sorted(glp.EXPORTS) == decl
    L = glp.lib()
    for name in decl:
        assert getattr(L, name) is not None
    assert L.glp_version() == 1


def test_status_strings():
    L = glp.lib()
    assert L.glp_status_string(0) == b"GLP_OK"
    assert L.glp_status_string(4) == b"GLP_ERR_WORKSPACE_TOO_SMALL"


def test_desc_validation():
    L = glp.lib()
    d = ctypes.c_void_p()
    assert L.glp_conv_desc_create(ctypes.byref(d), 0, 3, 8, 8, 4, 3, 3, 1, 1, 0, 0) == 1
    assert L.glp_conv_desc_create(ctypes.byref(d), 1, 3, 2, 2, 4, 3, 3, 1, 1, 0, 0) == 1  # H_o < 1
    assert L.glp_conv_desc_create(ctypes.byref(d), 1, 3, 8, 8, 4, 3, 3, 0, 1, 0, 0) == 1
    assert L.glp_conv_desc_create(ctypes.byref(d), 256, 3, 227, 227, 96, 11, 11, 4, 4, 0, 0) == 0
    ho, wo = ctypes.c_int(), ctypes.c_int()
    assert L.glp_conv_desc_get_output(d, ctypes.byref(ho), ctypes.byref(wo)) == 0
    assert (ho.value, wo.value) == (55, 55)
    assert L.glp_conv_desc_destroy(d) == 0


def test_plan_without_device_is_not_supported():
    import torch
    if torch.cuda.is_available():
        pytest.skip("device present")
    L = glp.lib()
    d = ctypes.c_void_p()
    assert L.glp_conv_desc_create(ctypes.byref(d), 2, 3, 8, 8, 4, 3, 3, 1, 1, 1, 1) == 0
    p = ctypes.c_void_p()
    assert L.glp_plan(ctypes.byref(p), d, 0, glp.GLP_MATH_BF16, 0) == 2   # NOT_SUPPORTED
    L.glp_conv_desc_destroy(d)
    with pytest.raises(glp.GlpError):
        glp.ConvLayer(2, 3, 8, 8, 4, 3, 1, 1)


def test_analyzer_paper_example_eq7():
    """P173 worked example through the product's Eq. 7 (K40C limits): 3."""
    lim = glp.DeviceLimits(15, 2048, 16, 65536, 48 * 1024, 0, 0, 32)
    assert glp.glp_analyze_eq7(lim, 512, 0, 18) == 3
    assert glp.glp_analyze_eq7(glp.glp_device_limits_b200(), 512, 0, 18) == 32


def test_b200_limits_match_north_star():
    lim = glp.glp_device_limits_b200()
    assert (lim.sm_count, lim.regs_per_sm, lim.smem_per_sm, lim.max_threads_per_sm,
            lim.max_blocks_per_sm, lim.tmem_cols_per_sm) == (148, 65536, 228 * 1024, 2048, 32, 512)


def test_ctas_per_sm_closed_form_vs_enumeration():
    """Product closed form == oracle enumeration over 3000 random kernel records."""
    lim = glp.glp_device_limits_b200()
    dev = A.B200()
    rnd = random.Random(7)
    for _ in range(3000):
        threads = rnd.choice([32, 64, 96, 128, 192, 256, 288, 384, 512, 768, 1024])
        regs = rnd.randint(16, 255)
        smem = rnd.choice([0, rnd.randint(0, 232448)])
        tmem = rnd.choice([0, 32, 64, 128, 256, 512])
        got = glp.glp_analyze_ctas_per_sm(lim, threads, regs, smem, tmem)
        exp = A.ctas_per_sm_enum(threads, regs, smem, tmem, dev)
        assert got == exp, (threads, regs, smem, tmem)


def test_samples_in_flight_vs_enumeration():
    rnd = random.Random(3)
    for _ in range(2000):
        slots, tps, n = rnd.randint(1, 1200), rnd.randint(1, 400), rnd.randint(1, 512)
        assert glp.glp_analyze_samples_in_flight(slots, tps, n) == A.samples_in_flight_enum(slots, tps, n)


def test_eq7_vs_oracle():
    lim = glp.glp_device_limits_b200()
    dev = A.B200()
    rnd = random.Random(5)
    for _ in range(1000):
        threads = rnd.choice([64, 128, 256, 512, 1024])
        smem = rnd.choice([0, 4096, 16384, 49152])
        blocks = rnd.randint(1, 5000)
        got = glp.glp_analyze_eq7(lim, threads, smem, blocks)
        exp = A.eq7_bound(A.Kernel(blocks=blocks, threads=threads, smem=smem), dev)
        assert got == exp


def test_plan_options_abi():
    """glp_plan_options_default fills the documented defaults; glp_plan_ex rejects an
    out-of-range option before touching a device (GLP_ERR_INVALID_VALUE)."""
    o = glp.plan_options()
    assert (o.cta_pairs, o.wgrad_cta_pairs, o.halo_wgrad, o.halo_fwd, o.halo_dgrad, o.fused_dy,
            o.fused_dy_builders, o.max_kblocks_per_stage, o.smem_cap) == (1, 1, 1, 1, 1, 1, 0, 4, 232448)
    L = glp.lib()
    d = ctypes.c_void_p()
    assert L.glp_conv_desc_create(ctypes.byref(d), 2, 3, 8, 8, 4, 3, 3, 1, 1, 1, 1) == 0
    p = ctypes.c_void_p()
    for bad in ({"halo_dgrad": 3}, {"max_kblocks_per_stage": 0}, {"wgrad_tile_n": 24},
                {"smem_cap": 1000}, {"wgrad_leaves": 3}):
        ob = glp.plan_options(**bad)
        assert L.glp_plan_ex(ctypes.byref(p), d, 0, glp.GLP_MATH_BF16, 0, ctypes.byref(ob)) == 1
    with pytest.raises(ValueError):
        glp.plan_options(no_such_option=1)
    L.glp_conv_desc_destroy(d)


def test_product_library_reads_no_environment():
    """The shipped library has no getenv: knobs are explicit plan options (glp_plan_ex), and
    the work-skipping diagnostics exist only in -DGLP_DIAG builds."""
    blob = open(glp.LIB_PATH, "rb").read()
    api = (b"GLP_OK", b"GLP_ERR_", b"GLP_PACK", b"GLP_PAC", b"GLP_MATH")   # enum names in messages
    knobs = sorted(k for k in set(re.findall(rb"GLP_[A-Z][A-Z0-9_]+", blob))
                   if not k.startswith(api))
    assert knobs == [], knobs


def test_tracker_exports_every_declared_symbol():
    """libglp_tracker.so (the CUPTI resource tracker, include/glp_tracker.h) loads and exports
    every declared call; its record structs match the header's field order."""
    from paper_conf_icpp_futhys18_b200 import tracker
    decl = header_functions("glp_tracker.h")
    assert sorted(tracker.EXPORTS) == decl
    L = tracker.lib()
    for name in decl:
        assert getattr(L, name) is not None
    src = open(os.path.join(ROOT, "include", "glp_tracker.h")).read()
    body = re.sub(r"/\*.*?\*/", "", src[src.index("typedef struct {"):src.index("} glp_kernel_record_t;")],
                  flags=re.S)
    fields = re.findall(r"\b(name|grid|block|cluster|regs|static_smem|dynamic_smem|queued_ns|"
                        r"submitted_ns|start_ns|end_ns|stream_id|correlation_id)\b", body)
    assert fields == [f for f, _ in tracker.KernelRecord._fields_]


def _header_struct_fields(header, typedef_name):
    """Field names of `typedef struct { ... } typedef_name;` in include/<header>, in order."""
    src = open(os.path.join(ROOT, "include", header)).read()
    end = src.index("} " + typedef_name + ";")
    start = src.rindex("typedef struct {", 0, end)
    body = re.sub(r"/\*.*?\*/", "", src[start + len("typedef struct {"):end], flags=re.S)
    names = []
    for decl in body.split(";"):
        decl = " ".join(decl.split())
        if not decl:
            continue
        decl = re.sub(r"^(unsigned |long long |long |const )*(int|size_t|double|float|long long|char)\b ?",
                      "", decl)
        names += [re.sub(r"\[.*\]", "", n).strip(" *") for n in decl.split(",")]
    return names


@pytest.mark.parametrize("typedef_name, cls", [
    ("glp_plan_info_t", glp.PlanInfo), ("glp_plan_options_t", glp.PlanOptions),
    ("glp_device_limits_t", glp.DeviceLimits), ("glp_kernel_attr_t", glp.KernelAttr)])
def test_binding_structs_match_header(typedef_name, cls):
    """The ctypes mirrors of the ABI structs list the header's fields in the header's order (a
    field added on one side only would shift every later field)."""
    assert _header_struct_fields("glp.h", typedef_name) == [f for f, _ in cls._fields_]
