"""The C-ABI library loads and exports every symbol include/h2tap.h declares (no GPU needed)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "h2tap.h")
LIB = os.path.join(ROOT, "paper_conf_edbt_jibrilabs23_b200", "libh2tap.so")


def declared_symbols():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(h2tap_[a-z_]+)\s*\(", text)))


@pytest.fixture(scope="module")
def lib():
    if not os.path.exists(LIB):
        subprocess.check_call(["make", "-C", ROOT, "lib"])
    return ctypes.CDLL(LIB)


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ("h2tap_replica_create_from_edges", "h2tap_replica_create_from_csr", "h2tap_delta_apply",
              "h2tap_replica_info", "h2tap_replica_export", "h2tap_bfs", "h2tap_sssp", "h2tap_pagerank", "h2tap_replica_liveness", "h2tap_delta_apply_records",
              "h2tap_replica_destroy", "h2tap_status_str", "h2tap_last_error"):
        assert s in syms


def test_library_exports_every_declared_symbol(lib):
    for s in declared_symbols():
        assert hasattr(lib, s), s
    out = subprocess.check_output(["nm", "-D", "--defined-only", LIB]).decode()
    exported = set(re.findall(r" T (h2tap_\w+)", out))
    assert set(declared_symbols()) <= exported


def test_host_only_entry_points(lib):
    lib.h2tap_version.restype = ctypes.c_char_p
    assert b"sm_100a" in lib.h2tap_version()
    lib.h2tap_status_str.restype = ctypes.c_char_p
    assert lib.h2tap_status_str(-5) == b"E_STALE_TS"
    assert lib.h2tap_status_str(0) == b"OK"
    # null handles are rejected without touching a device
    lib.h2tap_replica_info.restype = ctypes.c_int
    assert lib.h2tap_replica_info(None, None, None, None, None, None, None) == -1
    lib.h2tap_delta_apply.restype = ctypes.c_int
    assert lib.h2tap_delta_apply(None, None, ctypes.c_uint64(0), None) == -1


def test_collective_mode_host_entry_points(lib):
    """The collective mode's NCCL is loaded at run time: an id can be made on the host (no GPU),
    a too-small buffer is refused, and the per-replica stats refuse a null handle."""
    buf = ctypes.create_string_buffer(128)
    lib.h2tap_nccl_unique_id.restype = ctypes.c_int
    assert lib.h2tap_nccl_unique_id(buf, 128) == 0
    assert any(buf.raw)
    assert lib.h2tap_nccl_unique_id(buf, 16) == -1
    lib.h2tap_collective_stats.restype = ctypes.c_int
    assert lib.h2tap_collective_stats(None, None, None) == -1


def test_library_is_sm100a_code():
    out = subprocess.check_output(["cuobjdump", "--list-elf", LIB]).decode()
    assert "sm_100a" in out


def test_product_package_does_not_touch_the_oracle():
    pkg = os.path.join(ROOT, "paper_conf_edbt_jibrilabs23_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "o1_replay" not in src and "liboracle" not in src, f
                assert "o3_alg2" not in src and "libo3" not in src, f


def test_bench_dyn_gpu_measurement_does_not_touch_the_oracle():
    # only bench.py's cpu_baseline leg may run oracle/ code; bench_dyn.py is its GPU part
    src = open(os.path.join(ROOT, "bench_dyn.py")).read()
    assert "import oracle" not in src and "from oracle" not in src
