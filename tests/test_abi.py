"""CPU-side checks of the C-ABI library (no compute calls without a GPU).

* libfpx.so loads and exports every function include/fpx.h declares;
* the binding's enum values equal the header's;
* the header's record / entry layout agrees with the oracle's and the
  generator's own (independent) definitions;
* calls that must fail without touching the device do fail cleanly.
"""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

import fpxgen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "fpx.h")
LIB = os.path.join(ROOT, "paper_conf_hpdc_lilfslg23_b200", "libfpx.so")


def header_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(fpx_[a-z_0-9]+)\s*\(", src)) - {"fpx_entry", "fpx_options"})


def header_enums():
    src = re.sub(r"/\*.*?\*/", "", open(HEADER).read(), flags=re.S)
    vals = {}
    for m in re.finditer(r"\b(FPX_[A-Z0-9_]+)\s*=\s*(-?\d+)", src):
        vals[m.group(1)] = int(m.group(2))
    return vals


def test_library_exports_every_declared_symbol():
    funcs = header_functions()
    assert len(funcs) >= 16
    out = subprocess.run(["nm", "-D", "--defined-only", LIB], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (fpx_\w+)", out))
    missing = [f for f in funcs if f not in exported]
    assert not missing, missing
    L = ctypes.CDLL(LIB)
    for f in funcs:
        getattr(L, f)


def test_binding_names_match_header():
    from paper_conf_hpdc_lilfslg23_b200 import fpx

    assert sorted(fpx.EXPORTS) == header_functions()
    e = header_enums()
    for name, val in e.items():
        short = name[len("FPX_"):]
        if short.startswith("ERR_") or short in ("OK",):
            assert getattr(fpx, short) == val, name
        elif short in ("FP32", "FP64", "FP16", "BF16", "NAN", "INF", "SUB", "DIV0", "GEN", "PROP", "KILL",
                       "FLOW_NONE", "MODE_DEST", "MODE_FLOW", "FETCH_ALL", "FETCH_NEW", "OPT_SCAN_LDG", "OPT_NO_WARP_AGG", "OPT_LIVE_NEW", "OPT_STORM"):
            assert getattr(fpx, short) == val, name
    assert e["FPX_OP_COUNT"] == 20 and e["FPX_OP_DIV"] == 19 and e["FPX_OP_MUFU_RCP64H"] == 5


def test_layouts_agree_across_independent_definitions():
    from paper_conf_hpdc_lilfslg23_b200 import fpx

    assert fpx.lib.fpx_sizeof_rec_hdr() == oracle.lib().orc_sizeof_hdr() == fpxgen.lib().fpxgen_sizeof_hdr() == 16
    assert fpx.lib.fpx_sizeof_entry() == oracle.lib().orc_sizeof_entry() == 24
    assert fpx.ENTRY_DTYPE == oracle.ENTRY_DTYPE
    # key packing: site << 32 | fmt << 4 | flow << 2 | kind (FPX_KEY in the header)
    src = open(HEADER).read()
    assert "((uint64_t)(site) << 32) | ((uint64_t)(fmt) << 4) | ((uint64_t)(flow) << 2) | (uint64_t)(kind)" in src
    assert oracle.key(7, 3, 2, 1) == (7 << 32) | (3 << 4) | (2 << 2) | 1


def test_calls_without_device_fail_cleanly():
    from paper_conf_hpdc_lilfslg23_b200 import fpx

    h = ctypes.c_void_p()
    st = fpx.lib.fpx_open(0, None, ctypes.byref(h))
    assert st in (fpx.ERR_CUDA, fpx.ERR_INVALID, fpx.OK)
    if st == fpx.OK:  # a GPU is present: nothing to check here
        fpx.lib.fpx_close(h)
        return
    assert not h.value
    assert fpx.lib.fpx_open(0, None, None) == fpx.ERR_INVALID
    assert fpx.lib.fpx_scan_records(None, None, 1, None, 0, 0, 0, None) == fpx.ERR_INVALID
    assert fpx.lib.fpx_table_fetch(None, None, 0, None, 0) == fpx.ERR_INVALID
    assert fpx.lib.fpx_close(None) == fpx.ERR_INVALID
    assert fpx.lib.fpx_strerror(fpx.ERR_TABLE_FULL).startswith(b"exception table full")


def test_t4_summary_counts_distinct_sites():
    from paper_conf_hpdc_lilfslg23_b200 import fpx

    e = np.zeros(5, dtype=fpx.ENTRY_DTYPE)
    e["site"] = [1, 1, 2, 3, 3]
    e["fmt"] = [0, 0, 0, 1, 0]
    e["kind"] = [0, 0, 0, 2, 1]
    e["flow"] = [0, 1, 2, 0, 0]
    assert fpx.t4_summary(e) == {(0, 0): 2, (1, 2): 1, (0, 1): 1}


def test_report_lines_and_t4():
    from paper_conf_hpdc_lilfslg23_b200 import fpx, report

    e = np.zeros(4, dtype=fpx.ENTRY_DTYPE)
    e["site"] = [0x10002, 0x10002, 0x30001, 0x30001]
    e["fmt"] = [0, 0, 1, 1]
    e["kind"] = [0, 3, 1, 2]
    e["flow"] = [0, 0, 2, 3]
    e["count"] = [5, 1, 7, 2]
    e["first_index"] = [10, 11, 12, 13]
    names = {0x10002: ("ampere_sgemm_32x128_nn", "/unknown_path")}
    det = report.detector_lines(e, names)
    assert det[0].startswith("#GPU-FPX LOC-EXCEP INFO: in kernel [ampere_sgemm_32x128_nn], NaN found @ /unknown_path")
    assert det[0].endswith("[FP32] count=5 first=10") and "DIV0 found" in det[1] and len(det) == 2
    ana = report.analyzer_lines(e)
    assert ana[0].startswith("#GPU-FPX-ANA PROPAGATION: INF") and "[FP64]" in ana[0]
    assert ana[1].startswith("#GPU-FPX-ANA DISAPPEARANCE: SUB")
    assert report.t4_table(e) == {(0, 0): 1, (0, 3): 1, (1, 1): 1, (1, 2): 1}
    assert report.t4_lines(e)[1].split() == ["FP32", "1", "0", "0", "1"]


def test_selective_policy_is_alg3():
    import torch  # noqa: F401  (hooks imports torch)
    from paper_conf_hpdc_lilfslg23_b200.hooks import SelectivePolicy

    # no white-list, k = 0: every invocation (Alg3 lines 7-8)
    p = SelectivePolicy()
    assert all(p.should_scan("a") for _ in range(5))
    # white-list only (lines 3-6)
    p = SelectivePolicy(white_list={"a"})
    assert [p.should_scan(x) for x in "abab"] == [True, False, True, False]
    # 1 in k invocations per kernel, counted per name (lines 10-14)
    p = SelectivePolicy(k=3)
    assert [p.should_scan("a") for _ in range(7)] == [True, False, False, True, False, False, True]
    assert p.should_scan("b") and p.num == {"a": 7, "b": 1}
    p = SelectivePolicy(white_list={"a"}, k=2)
    assert [p.should_scan(x) for x in "aabba"] == [True, False, False, False, True]


def test_report_detail_states():
    from paper_conf_hpdc_lilfslg23_b200 import fpx, report

    e = np.zeros(2, dtype=fpx.ENTRY_DTYPE)
    e["site"] = [1, 2]
    e["flow"] = [2, 3]
    e["kind"] = [1, 0]
    e["detail"] = [2, 5]  # source 1 (fn4: INF flowed from R3); FSEL with a NaN source 0
    lines = report.analyzer_lines(e)
    assert lines[0].startswith("#GPU-FPX-ANA PROPAGATION: INF from source 1")
    assert lines[1].startswith("#GPU-FPX-ANA COMPARISON/DISAPPEARANCE: NaN from source 0")


def test_header_is_plain_c_and_links(tmp_path):
    """include/fpx.h is a C header: a C99 program (-pedantic, warnings as
    errors) includes it, links libfpx.so and calls an entry point that needs
    no GPU."""
    import shutil

    if shutil.which("gcc") is None:
        pytest.skip("no gcc")
    libdir = os.path.dirname(LIB)
    src = tmp_path / "t.c"
    src.write_text('#include "fpx.h"\n#include <stdio.h>\n'
                   "int main(void) {\n  fpx_handle h = 0;\n  fpx_options o = {0, 0, 0};\n"
                   "  fpx_rec_hdr r = {1u, 0xFFFFFFFFu, 0u, 0u};\n  (void)h; (void)o; (void)r;\n"
                   '  printf("%s|%s\\n", fpx_strerror(FPX_OK), fpx_strerror(FPX_ERR_TABLE_FULL));\n'
                   "  return (int)sizeof(fpx_entry) - 24;\n}\n")
    exe = tmp_path / "t"
    subprocess.run(["gcc", "-std=c99", "-Wall", "-Wextra", "-pedantic", "-Werror", "-I", os.path.dirname(HEADER),
                    str(src), "-L", libdir, "-lfpx", f"-Wl,-rpath,{libdir}", "-o", str(exe)], check=True)
    out = subprocess.run([str(exe)], capture_output=True, text=True)
    assert out.returncode == 0, out.stderr
    a, b = out.stdout.strip().split("|")
    assert a and b and a != b


def test_shared_tables_use_system_scope_atomics():
    """A table shared across GPUs (fpx_table_export / fpx_open_attached) is
    updated from several devices at once: the library carries system-scope
    CAS / ADD / MIN for it next to the device-scope ones of local tables
    (CUDA memory model: an atomic is atomic only within its scope)."""
    sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True, check=True).stdout
    for op in ("CAS", "ADD", "MIN"):
        # ATOM (value returned) or REDG (fire-and-forget reduction)
        assert re.search(rf"(ATOMG?|REDG)\.E\.{op}\.64\.STRONG\.SYS", sass), op
        assert re.search(rf"(ATOMG?|REDG)\.E\.{op}\.64\.STRONG\.GPU", sass), op
