"""CPU-only: the C-ABI library builds, loads, and exports every symbol that
include/rcm.h declares (no compute calls: there is no GPU here)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "rcm.h")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(rcm_[a-z_]+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = _declared()
    for f in ["rcm_plan_create", "rcm_reorder", "rcm_reorder_batched", "rcm_sync_status",
              "rcm_get_stats", "rcm_plan_destroy", "rcm_status_string", "rcm_find_pseudo_peripheral"]:
        assert f in names


def test_library_exports_every_declared_symbol():
    import paper_conf_ipps_mlakarwps21_b200 as rcm
    lib = ctypes.CDLL(rcm.LIB_PATH)
    for name in _declared():
        assert hasattr(lib, name), name
    assert sorted(rcm.EXPORTS) == _declared()
    out = subprocess.run(["nm", "-D", "--defined-only", rcm.LIB_PATH], capture_output=True, text=True).stdout
    for name in _declared():
        assert re.search(rf"\bT {name}$", out, flags=re.M), name


def test_host_only_entry_points():
    import paper_conf_ipps_mlakarwps21_b200 as rcm
    assert rcm.rcm_status_string(0) == "ok"
    assert rcm.rcm_status_string(5).startswith("queue")
    o = rcm.rcm_default_options(batch_nodes=64)
    assert o.batch_nodes == 64 and o.temp_elems == 0 and o.flags == 0


def test_library_is_sm100a():
    import paper_conf_ipps_mlakarwps21_b200 as rcm
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", rcm.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_oracle_and_product_share_no_code():
    """Neither side imports / includes / links the other."""
    prod = os.path.join(ROOT, "paper_conf_ipps_mlakarwps21_b200")
    pat_prod = re.compile(r"^\s*(import\s+oracle|from\s+oracle|#\s*include\s+.*oracle)", re.M)
    for dirpath, _, files in os.walk(prod):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                assert not pat_prod.search(open(os.path.join(dirpath, f)).read()), f
    pat_orc = re.compile(r"^\s*(import\s+paper_conf|from\s+paper_conf|#\s*include\s+.*(rcm\.h|csrc))", re.M)
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c", ".h")):
            assert not pat_orc.search(open(os.path.join(ROOT, "oracle", f)).read()), f
