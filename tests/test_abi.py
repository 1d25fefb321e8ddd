"""The C-ABI library builds, loads and exports every symbol include/mm.h
declares (no compute calls: this runs on CPU-only hosts too)."""
import ctypes
import os
import re
import subprocess

import pytest

from conftest import ROOT, gpu_available

HEADER = os.path.join(ROOT, "include", "mm.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"^\s*(?:int|const char\s*\*)\s*(mm_\w+)\s*\(", src, flags=re.M)
    return sorted(set(names))


def test_header_declares_the_north_star_calls():
    names = declared_functions()
    for n in ["mm_create", "mm_post_recvs", "mm_push_msgs", "mm_match_batch", "mm_destroy"]:
        assert n in names


def test_library_builds_and_exports_every_declared_symbol():
    from paper_conf_ipps_klenkfed17_b200 import _build, _lib
    path = _build.build_library()
    out = subprocess.run(["nm", "-D", "--defined-only", path], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (mm_\w+)", out))
    for n in declared_functions():
        assert n in exported, n
        assert n in _lib.SIGNATURES, "binding lacks " + n
    L = _lib.load()
    for n in declared_functions():
        assert getattr(L, n) is not None


def test_library_is_sm100a():
    from paper_conf_ipps_klenkfed17_b200 import _build
    out = subprocess.run(["cuobjdump", "--list-elf", _build.build_library()], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def test_strerror_and_version():
    from paper_conf_ipps_klenkfed17_b200 import _lib
    L = _lib.load()
    assert L.mm_version().decode().startswith("mm ")
    assert L.mm_strerror(3).decode() == "queue or output capacity exceeded"


def test_argument_errors_without_device():
    from paper_conf_ipps_klenkfed17_b200 import _lib
    L = _lib.load()
    h = ctypes.c_void_p()
    assert L.mm_create(None, 0, 1, 4, 4, None) == _lib.MM_ERR_ARG
    assert L.mm_create(ctypes.byref(h), 7, 1, 4, 4, None) == _lib.MM_ERR_ARG
    assert L.mm_create(ctypes.byref(h), 1, 2, 4, 4, None) == _lib.MM_ERR_ARG  # no-wildcard: one endpoint
    assert L.mm_create(ctypes.byref(h), 0, 1, 4, 1 << 20, None) == _lib.MM_ERR_ARG  # > MM_MPI_MAX_MSGS
    assert L.mm_post_recvs(None, None, None, None, 0) == _lib.MM_ERR_ARG
    assert L.mm_match_batch(None, None, None, 0, None) == _lib.MM_ERR_ARG
    assert L.mm_destroy(None) == _lib.MM_OK
    assert L.mm_route(None, None, 0, 0, 0, 0, None, None, None, None) == _lib.MM_ERR_ARG


@pytest.mark.skipif(gpu_available(), reason="checks the no-device path")
def test_no_device_fails_loudly():
    from paper_conf_ipps_klenkfed17_b200 import Engine, MMError
    with pytest.raises(MMError):
        Engine(0, 1, 16, 16)


def header_constants():
    """NAME = value pairs of the enums and #defines in include/mm.h."""
    src = re.sub(r"/\*.*?\*/", "", open(HEADER).read(), flags=re.S)
    vals = {}
    for body in re.findall(r"enum\s*\w*\s*\{(.*?)\}", src, flags=re.S):
        nxt = 0
        for item in [x.strip() for x in body.split(",") if x.strip()]:
            m = re.match(r"(\w+)\s*(?:=\s*(-?\w+))?", item)
            name, v = m.group(1), m.group(2)
            nxt = int(v, 0) if v is not None else nxt
            vals[name] = nxt
            nxt += 1
    for name, v in re.findall(r"#define\s+(MM_\w+)\s+\(?(-?(?:0x)?[0-9A-Fa-f]+)[uUlL]*\)?", src):
        vals[name] = int(v, 0)
    return vals


def test_binding_constants_match_the_header():
    """Every MM_* constant the Python binding defines has the header's value
    (options, query slots, semantics levels, error codes, wildcards)."""
    from paper_conf_ipps_klenkfed17_b200 import _lib
    hdr = header_constants()
    mine = {k: getattr(_lib, k) for k in dir(_lib) if k.startswith("MM_") and isinstance(getattr(_lib, k), int)}
    common = sorted(set(hdr) & set(mine))
    for k in ["MM_OPT_PIPELINE_CHUNKS", "MM_Q_FALLBACKS", "MM_Q_COUNT", "MM_SEM_MPI", "MM_OPT_MPI_KERNEL"]:
        assert k in common, k
    for k in common:
        assert hdr[k] == mine[k], (k, hdr[k], mine[k])
