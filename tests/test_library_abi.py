"""CPU-side checks of the boundary: libigd.so builds for sm_100a, loads, and exports every
symbol include/igd.h declares (no compute calls: there is no GPU here)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "igd.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:const\s+)?[\w\s\*]+?\b(igd_\w+)\s*\(", src, flags=re.M)
    return sorted(set(n for n in names if not n.endswith("_fn")))


def test_header_declares_the_north_star_calls():
    names = declared_functions()
    for required in ("igd_ctx_create", "igd_trace_load", "igd_detect", "igd_reports", "igd_ctx_destroy",
                     "igd_strerror"):
        assert required in names


def test_library_exports_every_declared_symbol():
    import paper_conf_sosp_kamathb21_b200 as igd

    lib = igd.load_library()
    for name in declared_functions():
        assert hasattr(lib, name), name
    out = subprocess.check_output(["nm", "-D", "--defined-only", igd.lib_path()]).decode()
    for name in declared_functions():
        assert re.search(rf"\bT {name}\b", out), f"{name} not exported"


def test_library_is_sm100a():
    import paper_conf_sosp_kamathb21_b200 as igd

    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", igd.lib_path()]).decode()
    assert "sm_100a" in out


def test_strerror_and_argument_errors_without_gpu():
    import paper_conf_sosp_kamathb21_b200 as igd

    lib = igd.load_library()
    assert lib.igd_strerror(-2).decode() == "ill-formed trace event"
    # NULL out-pointer is rejected before any CUDA call
    assert lib.igd_ctx_create(None, 0, None, 1, 0, None, igd.igd.ALLOC_FN(), igd.igd.FREE_FN(), None) == -1
    assert lib.igd_detect(None, 0, None) == -1
    assert lib.igd_bad_event(None) == 0


def test_struct_sizes_match_header():
    import paper_conf_sosp_kamathb21_b200 as igd

    assert igd.EVENT_DTYPE.itemsize == 16 and igd.REPORT_DTYPE.itemsize == 32
    assert ctypes.sizeof(igd.igd.igd_trace_desc) == 40


def test_product_does_not_import_oracle():
    # the product path never imports, links or includes the oracle (it is test infrastructure)
    pkg = os.path.join(ROOT, "paper_conf_sosp_kamathb21_b200")
    for dp, _, files in os.walk(pkg):
        for f in files:
            path = os.path.join(dp, f)
            if f.endswith(".py"):
                txt = open(path).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", txt, flags=re.M), f
                assert "igd_oracle" not in txt and "libigd_oracle" not in txt, f
            if f.endswith((".cu", ".cuh", ".h")):
                txt = open(path).read()
                assert not re.search(r"#include\s+[\"<].*oracle", txt), f
                assert "igdo_" not in txt, f


def test_nccl_unique_id_without_gpu():
    # the multi-GPU boundary: libnccl is resolved at run time and an id is 128 bytes
    import paper_conf_sosp_kamathb21_b200 as igd

    a, b = igd.igd_nccl_unique_id(), igd.igd_nccl_unique_id()
    assert len(a) == 128 and len(b) == 128 and a != b


def test_collective_create_argument_errors_without_gpu():
    import paper_conf_sosp_kamathb21_b200 as igd

    lib = igd.load_library()
    ctx = ctypes.c_void_p()
    A, F = igd.igd.ALLOC_FN(), igd.igd.FREE_FN()
    assert lib.igd_ctx_create(ctypes.byref(ctx), 0, None, 2, 0, None, A, F, None) == -1  # nranks > 1, no id
    assert lib.igd_ctx_create(ctypes.byref(ctx), 0, None, 2, 2, None, A, F, None) == -1  # rank out of range
    assert lib.igd_ctx_create(ctypes.byref(ctx), 0, None, 0, 0, None, A, F, None) == -1  # no ranks
