"""CPU-side checks of the boundary: the C-ABI library builds, loads without a GPU and
exports every function include/sptrsv.h declares; the binding's marshalling tables
match the header.  No compute calls (no GPU here)."""
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "sptrsv.h")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(sptrsv_[a-z_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def libpath():
    import __graft_entry__
    return __graft_entry__._load_builder().build()


def test_header_declares_the_north_star_entry_points():
    d = _declared()
    for name in ("sptrsv_analyse_csr", "sptrsv_solve", "sptrsv_destroy"):
        assert name in d


def test_library_exports_every_declared_symbol(libpath):
    out = subprocess.run(["nm", "-D", "--defined-only", libpath], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT\s+(sptrsv_[a-z_]+)\b", out))
    missing = [f for f in _declared() if f not in exported]
    assert not missing, missing


def test_binding_covers_header_and_loads(libpath):
    import paper_conf_icpp_suz0hw0w20_b200._lib as L
    assert sorted(L.EXPORTS) == _declared()
    assert L.lib.sptrsv_abi_version() == 4
    assert L.lib.sptrsv_strerror(-3).decode().startswith("row without a diagonal")
    # argument validation happens before any CUDA call
    assert L.lib.sptrsv_analyse_csr(-1, None, None, None, None) == L.ERR_INVALID_ARG
    assert L.lib.sptrsv_solve(None, None, None, None) == L.ERR_INVALID_ARG
    assert L.lib.sptrsv_destroy(None) == L.OK


def test_status_codes_match_oracle_numbering():
    import oracle
    import paper_conf_icpp_suz0hw0w20_b200._lib as L
    for name in ("NOT_LOWER", "MISSING_DIAG", "ZERO_DIAG", "BAD_ROWPTR", "BAD_COL"):
        assert getattr(oracle, name) == getattr(L, "ERR_" + name)
    assert oracle.UNSORTED == L.ERR_UNSORTED


def test_kernels_are_sm100a_sass(libpath):
    out = subprocess.run(["cuobjdump", "--list-elf", libpath], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    sass = subprocess.run(["cuobjdump", "-sass", libpath], capture_output=True, text=True).stdout
    # the flag protocol: acquire polls (strong GPU loads + L1 invalidate), release publishes
    assert "LDG.E.STRONG.GPU" in sass and "CCTL.IVALL" in sass and "NANOSLEEP" in sass


def test_product_package_never_imports_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icpp_suz0hw0w20_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "oracle.c" not in txt, f


def test_only_tests_smoke_and_bench_touch_the_oracle():
    """The oracle is test infrastructure: outside tests/, only __graft_entry__.smoke() and
    bench.py's cpu_baseline / reference legs may import it (tools/, synth/ and include/ never do)."""
    for sub in ("tools", "synth", "include"):
        for dp, _, fs in os.walk(os.path.join(ROOT, sub)):
            for f in fs:
                if f.endswith((".py", ".cu", ".cuh", ".h", ".c")):
                    txt = open(os.path.join(dp, f)).read()
                    assert "import oracle" not in txt and "from oracle" not in txt, os.path.join(dp, f)


def test_reference_arm_loads_no_product_library():
    """bench.py --impl reference runs the oracle only: the product package (and libsptrsv.so)
    must not be imported, so the driver's native-library census of that arm lists oracle/ alone."""
    code = ("import sys, bench; a = bench.parse(['--impl', 'reference', '--config', 'c1', '--steps', '2', "
            "'--warmup', '1']); bench.run_reference(a, 0, 1); "
            "assert not any(m.startswith('paper_conf_icpp_suz0hw0w20_b200') for m in sys.modules), 'product imported'; "
            "import os; maps = open('/proc/self/maps').read(); assert 'libsptrsv' not in maps")
    r = subprocess.run(["python", "-c", code], cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    line = [l for l in r.stdout.splitlines() if l.startswith("{")][-1]
    import json
    d = json.loads(line)
    assert d["impl"] == "reference" and d["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 0


def test_bench_defaults():
    import sys
    sys.path.insert(0, ROOT)
    import bench
    assert bench.parse([]).config == "c2" and bench.parse([]).gpus == 1
    assert bench.parse(["--gpus", "4"]).config == "c2"  # N > 1: c2 on every GPU (weak) + the C5 leg
    a = bench.parse(["--gpus", "2", "--config", "c2"])
    assert a.config == "c2"
