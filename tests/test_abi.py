"""CPU-side checks of the boundary: the C-ABI library builds/loads and exports
every function include/eirene.h declares (no compute calls without a GPU)."""
import ctypes
import os
import subprocess

import pytest

from paper_conf_ppopp_zhangz0lzl23_b200 import _ffi
from paper_conf_ppopp_zhangz0lzl23_b200.build import LIB, build


@pytest.fixture(scope="module")
def libpath():
    return build()


def test_library_exports_every_header_symbol(libpath):
    names = _ffi.header_functions()
    assert len(names) >= 14
    L = ctypes.CDLL(libpath)
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing, f"missing exports: {missing}"
    # the binding declares a signature for every header function, and nothing else
    assert sorted(_ffi._SIGS) == names


def test_exports_are_c_linkage(libpath):
    out = subprocess.run(["nm", "-D", "--defined-only", libpath], capture_output=True, text=True).stdout
    exported = {line.split()[-1] for line in out.splitlines() if " T " in line}
    for n in _ffi.header_functions():
        assert n in exported, n


def test_key32_library_exports_the_same_abi(libpath):
    """libeirene32.so (-DEIRENE_KEY32) exports the same C ABI
    with 32-bit keys / values; it builds for sm_100a only."""
    from paper_conf_ppopp_zhangz0lzl23_b200.build import build_all
    p32 = build_all()[1]
    assert p32.endswith("libeirene32.so")
    L = ctypes.CDLL(p32)
    assert not [n for n in _ffi.header_functions() if not hasattr(L, n)]
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", p32], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    L32 = _ffi.lib(32)
    h = ctypes.c_void_p()
    cfg = _ffi.eirene_config()
    L32.eirene_default_config(ctypes.byref(cfg))
    cfg.key_lo = 1 << 32   # no 32-bit key lies at or above 2^32 - 1
    assert L32.eirene_create(ctypes.byref(cfg), ctypes.byref(h)) == _ffi.EIRENE_EINVAL


def test_sm100a_code_only(libpath):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", libpath], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out
    for other in ("sm_80", "sm_90"):
        assert other + "." not in out


def test_host_only_calls_without_gpu(libpath):
    L = _ffi.lib()
    cfg = _ffi.eirene_config()
    L.eirene_default_config(ctypes.byref(cfg))
    assert cfg.fanout == 16 and cfg.max_batch == 1 << 20 and cfg.retry_threshold == 4
    assert cfg.key_hi == (1 << 64) - 1
    assert L.eirene_strerror(_ffi.EIRENE_EFULL).decode().startswith("node pools")
    # argument validation happens before any device call
    h = ctypes.c_void_p()
    bad = _ffi.eirene_config()
    L.eirene_default_config(ctypes.byref(bad))
    bad.fanout = 8
    assert L.eirene_create(ctypes.byref(bad), ctypes.byref(h)) == _ffi.EIRENE_EINVAL
    assert L.eirene_create(None, ctypes.byref(h)) == _ffi.EIRENE_EINVAL
    assert L.eirene_results(None, 1, None) == _ffi.EIRENE_EINVAL
    assert L.eirene_destroy(None) == _ffi.EIRENE_EINVAL


def test_product_package_never_imports_oracle():
    root = os.path.dirname(_ffi.PKG)
    pkg = _ffi.PKG
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                text = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in text and "from oracle" not in text, f
                assert "eirene_oracle" not in text, f
    # the oracle includes nothing from the product
    for f in os.listdir(os.path.join(root, "oracle")):
        if f.endswith((".cpp", ".h")):
            text = open(os.path.join(root, "oracle", f)).read()
            assert "eirene.h\"" not in text.replace("eirene_oracle.h\"", "") and "csrc" not in text.split("*/")[-1]


def test_range_and_prepare_argument_checks_without_gpu(libpath):
    """The range entry point and the graph warm-up validate their arguments on
    the host (EINVAL) before touching the device."""
    L = _ffi.lib()
    tk = ctypes.c_uint64()
    assert L.eirene_submit_batch_range(None, None, None, None, 1, None, 8, None, None, None,
                                       ctypes.byref(tk)) == _ffi.EIRENE_EINVAL
    assert L.eirene_prepare_batch(None, 16, 0) == _ffi.EIRENE_EINVAL
    assert _ffi.EIRENE_RANGE == 4


def test_probe_gather_argument_checks(libpath):
    """eirene_probe_gather validates its arguments before any device call."""
    L = _ffi.lib()
    assert L.eirene_probe_gather(None, 1 << 20, 16, 0, 1, None) == _ffi.EIRENE_EINVAL
    assert L.eirene_probe_gather(ctypes.c_void_p(1 << 20), 1024, 16, 0, 1, None) == _ffi.EIRENE_EINVAL   # short
    assert L.eirene_probe_gather(ctypes.c_void_p((1 << 20) + 8), 1 << 20, 16, 0, 1, None) == _ffi.EIRENE_EINVAL
    assert L.eirene_probe_gather(ctypes.c_void_p(1 << 20), 1 << 20, 16, 4, 1, None) == _ffi.EIRENE_EINVAL   # kind
    assert L.eirene_probe_gather(ctypes.c_void_p(1 << 20), 3 << 20, 16, 0, 1, None) == _ffi.EIRENE_EINVAL   # not 2^k


def test_fused_routing_argument_checks_without_gpu(libpath):
    """The fused-routing calls reject a null handle or null outputs on the host (EINVAL)
    before touching the device; the IPC handle size is the header's."""
    L = _ffi.lib()
    addr = ctypes.c_void_p()
    n = ctypes.c_uint32()
    inv = ctypes.c_uint32()
    E = _ffi.EIRENE_EINVAL
    assert L.eirene_route_arena_create(None, 2, 0, 1024, ctypes.byref(addr), None) == E
    assert L.eirene_route_arena_open_ipc(None, None, ctypes.byref(addr)) == E
    assert L.eirene_route_arena_connect(None, None) == E
    assert L.eirene_route_push(None, None, None, None, 0, None, None, None) == E
    assert L.eirene_route_pull(None, None, None, None, 0, ctypes.byref(n), ctypes.byref(inv), None) == E
    assert L.eirene_route_push_results(None, None, None) == E
    assert L.eirene_route_unpermute_arena(None, None, 0, None, None) == E
    with open(_ffi.HEADER) as f:
        assert "#define EIRENE_IPC_HANDLE_BYTES 64" in f.read()
    assert _ffi.EIRENE_IPC_HANDLE_BYTES == 64
