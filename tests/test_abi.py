"""C-ABI library: loads without a GPU, exports every symbol include/mapsm.h
declares, and its pure-host entry points behave (no compute calls here)."""
import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "mapsm.h")


def declared_symbols():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(mapsm_[a-z0-9_]+)\s*\(", text)))


def test_header_declares_the_north_star_calls():
    syms = declared_symbols()
    for s in ["mapsm_grid_create", "mapsm_window_set", "mapsm_iterate", "mapsm_gather", "mapsm_bind",
              "mapsm_sync", "mapsm_plan_query"]:
        assert s in syms


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(M._LIB_PATH)
    for s in declared_symbols():
        assert hasattr(lib, s), s
    out = subprocess.check_output(["nm", "-D", "--defined-only", M._LIB_PATH]).decode()
    exported = set(re.findall(r" T (mapsm_\w+)", out))
    assert set(declared_symbols()) <= exported
    assert set(M.EXPORTED) == set(declared_symbols())


def test_library_is_sm100a_only():
    out = subprocess.check_output(["cuobjdump", "--list-elf", M._LIB_PATH]).decode()
    assert "sm_100a" in out
    for other in ["sm_90", "sm_80", "sm_103"]:
        assert other + "." not in out and other + "a." not in out


def test_status_strings_and_version():
    L = M.lib()
    assert L.mapsm_status_string(0) == b"MAPSM_OK"
    assert L.mapsm_status_string(-5) == b"MAPSM_ESTATE"
    assert b"sm_100a" in L.mapsm_version()


def test_null_and_bad_arguments_fail_cleanly():
    L = M.lib()
    assert L.mapsm_iterate(None, 1) == M.EINVAL
    assert L.mapsm_grid_destroy(None) == M.EINVAL
    assert L.mapsm_ctx_destroy(None) == M.EINVAL
    assert b"NULL" in L.mapsm_last_error()
    with pytest.raises(M.MapsmError) as e:
        M.mapsm_plan_query(10, 0, 1, M.WRAP, 0)
    assert e.value.status == M.EINVAL


def test_no_cpu_fallback_symbols():
    """The product library contains no host implementation of the stencil: its
    only compute entry points launch kernels (cuobjdump lists them)."""
    out = subprocess.check_output(["cuobjdump", "--list-text", M._LIB_PATH]).decode()
    assert "life_step_kernel" in out and "conv_step_kernel" in out
    assert "pack_life_kernel" in out and "unpack_life_kernel" in out


def test_binding_constants_match_header_enums():
    """Every MAPSM_* enumerator of include/mapsm.h that the binding mirrors
    (same name without the prefix) has the same value in mapsm.py."""
    import re

    from paper_conf_sc_ben_nunlbr15_b200 import mapsm as M

    text = open(os.path.join(ROOT, "include", "mapsm.h")).read()
    body = " ".join(re.findall(r"typedef enum\s*\{(.*?)\}", text, re.S))
    enums = {k: int(v) for k, v in re.findall(r"MAPSM_([A-Z0-9_]+)\s*=\s*(-?\d+)", body)}
    assert len(enums) > 40
    aliases = {"LIFE_REG": "KERNEL_LIFE_REG"}
    checked = 0
    for name, value in enums.items():
        py = name if hasattr(M, name) else aliases.get(name)
        if py is None or not hasattr(M, py):
            continue
        assert getattr(M, py) == value, (name, getattr(M, py), value)
        checked += 1
    for must in ("OPT_EXCHANGE_SMS", "OPT_HOST_PACKED", "EXCHANGE_CE", "KERNEL_CONV_TB2", "OPT_DEEP_HALO"):
        assert must in enums and getattr(M, must) == enums[must], must
    assert checked >= 25, checked
