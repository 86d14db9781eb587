"""CPU checks of the C-ABI library (``-m "not gpu"``): it builds for sm_100a,
loads without a GPU, exports every symbol include/hpccg.h declares, the
ctypes layout of hpccg_stats matches the header, the SASS is sm_100a, and
error paths return codes instead of crashing.  No compute calls."""
import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_sc_valero_laragmtv24_b200 import _build
from paper_conf_sc_valero_laragmtv24_b200 import hpccg as H


@pytest.fixture(scope="module")
def lib():
    _build.build()
    return H.lib()


def test_exports_every_header_symbol(lib):
    syms = H.header_symbols()
    assert len(syms) >= 20
    out = subprocess.run(["nm", "-D", "--defined-only", H.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT (hpccg_\w+)", out))
    missing = [s for s in syms if s not in exported]
    assert not missing, missing
    extra = sorted(exported - set(syms))
    assert not extra, f"exported but not declared: {extra}"
    assert set(H._SIGS) == set(syms), "binding signatures out of sync with header"


def test_stats_struct_layout_matches_header():
    txt = open(H.HEADER).read()
    body = re.search(r"typedef struct hpccg_stats \{(.*?)\} hpccg_stats;", txt, re.S).group(1)
    fields = re.findall(r"(double|int64_t)\s+(\w+);", body)
    assert [f for _, f in fields] == [f for f, _ in H.hpccg_stats._fields_]
    assert ctypes.sizeof(H.hpccg_stats) == 8 * len(fields)


def test_header_constants_match_binding():
    txt = open(H.HEADER).read()
    consts = dict((k, int(v)) for k, v in re.findall(r"#define (HPCCG_\w+) \(?(-?\d+)\)?", txt))
    for k, v in consts.items():
        assert getattr(H, k) == v, k


def test_strings_without_gpu(lib):
    assert "sm_100a" in H.hpccg_version()
    assert H.hpccg_strerror(H.HPCCG_EINVAL) == "HPCCG_EINVAL"
    assert H.hpccg_strerror(-99) == "HPCCG_E?"


def test_error_codes_not_crashes(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("checks the no-GPU error path")
    with pytest.raises(H.HpccgError) as e:
        H.hpccg_init(0)
    assert e.value.code == H.HPCCG_ECUDA
    with pytest.raises(H.HpccgError) as e:
        H.hpccg_init(0, nranks=0)
    assert e.value.code == H.HPCCG_EINVAL
    # NULL handles are rejected, not dereferenced
    assert lib.hpccg_solve(None, 10, 0.0, None, None, None) == H.HPCCG_EINVAL
    assert lib.hpccg_ddot(None, 0, None, None, None) == H.HPCCG_EINVAL
    assert lib.hpccg_info(None, None, None, None, None, None) == H.HPCCG_EINVAL


def test_sass_is_sm100a_and_fp64(lib):
    cuobjdump = "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(cuobjdump):
        pytest.skip("no cuobjdump")
    out = subprocess.run([cuobjdump, "-lelf", H.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run([cuobjdump, "-sass", H.LIB_PATH], capture_output=True,
                          text=True).stdout
    funcs = re.split(r"\n\s+Function : ", sass)
    spmv = [f for f in funcs if f.startswith("_ZN5hpccg13spmv27_kernel")]
    assert spmv and all("DFMA" in f for f in spmv)   # fp64 FMA chain
    assert "HMMA" not in sass and "UTCHMMA" not in sass  # no tensor cores (HBM-bound path)


def test_product_does_not_import_oracle():
    """The product package never imports / links / executes oracle/."""
    pkg = os.path.dirname(H.__file__)
    for root, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(root, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", src, re.M), f
                assert "hpccg_oracle" not in src and "liboracle" not in src, f


def test_no_readonly_loads_ahead_of_the_pdl_wait(lib):
    """PDL safety (structural): in every kernel that waits on its predecessor
    (griddepcontrol.wait = SASS ACQBULK), no read-only-path load of anything
    but the matrix stream (LDG ... .NA ... .CONSTANT = ld.global.nc
    L1::no_allocate) may come before the first wait.  Device scalars and
    partial sums are read with ordered loads (kernels.cuh ldg_o) so the
    compiler cannot hoist them above it (an __ldg may legally move)."""
    cuobjdump = "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(cuobjdump):
        pytest.skip("no cuobjdump")
    sass = subprocess.run([cuobjdump, "-sass", H.LIB_PATH], capture_output=True, text=True).stdout
    funcs = re.split(r"\n\s+Function : ", sass)[1:]
    waiting = [f for f in funcs if "ACQBULK" in f]
    assert len(waiting) > 20
    bad = []
    for f in waiting:
        pre = f.split("ACQBULK")[0]
        loads = set(re.findall(r"LDG\.E[A-Z0-9._]*", pre))
        early = sorted(x for x in loads if "CONSTANT" in x and ".NA." not in x)
        if early:
            bad.append((f.split("\n", 1)[0][:80], early))
    assert not bad, bad


# The product kernels of the CG loop must not spill (ptxas -v in the build
# log): two regressions of this kind were each worth 2.7-4.6 % of their
# kernel (a field inserted into SpmvArgs, a live ring pointer in the fused
# z-slab SpMV).
NO_SPILL = [
    "_ZN5hpccg15spmv27x2_kernelILi1ELb0ELb0ELb0ELb0EEEvNS_8SpmvArgsE",   # single slab, plain / per-iteration graph
    "_ZN5hpccg15spmv27x2_kernelILi1ELb1ELb0ELb0ELb0EEEvNS_8SpmvArgsE",   # single slab, while-graph (U > 1)
    "_ZN5hpccg15spmv27x2_kernelILi1ELb0ELb1ELb0ELb0EEEvNS_8SpmvArgsE",   # z-slabs (HALO_PEER 2)
    "_ZN5hpccg15spmv27x2_kernelILi1ELb1ELb1ELb0ELb0EEEvNS_8SpmvArgsE",
    "_ZN5hpccg15spmv27x2_kernelILi1ELb0ELb1ELb0ELb1EEEvNS_8SpmvArgsE",   # z-slabs with the p ring
    "_ZN5hpccg15spmv27x2_kernelILi1ELb1ELb1ELb0ELb1EEEvNS_8SpmvArgsE",
    "_ZN5hpccg15spmv27x2_kernelILi1ELb0ELb0ELb0ELb1EEEvNS_8SpmvArgsE",   # single slab with the p ring
    "_ZN5hpccg22cg_pupdate_ring_kernelILi4ELb0EEEvNS_9PringArgsE",
    "_ZN5hpccg22cg_pupdate_ring_kernelILi4ELb1EEEvNS_9PringArgsE",
    "_ZN5hpccg18cg_pupdate1_kernelILi4ELb0EEEvNS_9Pupd1ArgsE",
    "_ZN5hpccg17cg_update1_kernelILi4ELb0ELb0EEEvNS_8Upd1ArgsE",
    "_ZN5hpccg17cg_update1_kernelILi4ELb1ELb0EEEvNS_8Upd1ArgsE",
    "_ZN5hpccg22cg_smem_cluster_kernelILi512ELb0ELb0ELb1EEEvNS_8SmemArgsE",  # on chip, configs[0]
    "_ZN5hpccg22cg_smem_cluster_kernelILi512ELb0ELb0ELb0EEEvNS_8SmemArgsE",
    "_ZN5hpccg23tri_pupdate_ring_kernelElPKdPdNS_7TriRingEPKNS_10TriScalarsE",
]


def test_product_kernels_do_not_spill(lib):
    log = os.path.join(os.path.dirname(H.LIB_PATH), "build.log")
    if not os.path.exists(log):
        pytest.skip("no build log (library built elsewhere)")
    txt = open(log).read()
    spills = {}
    for m in re.finditer(r"Compiling entry function '(\w+)' for 'sm_100a'\n.*?\n\s*(\d+) bytes stack frame, "
                         r"(\d+) bytes spill stores", txt):
        spills[m.group(1)] = int(m.group(3))
    missing = [k for k in NO_SPILL if k not in spills]
    assert not missing, missing
    bad = {k: spills[k] for k in NO_SPILL if spills[k]}
    assert not bad, bad
