"""The C-ABI library loads and exports every symbol include/*.h declares;
host-only logic (partitioner) agrees with the oracle.  CPU only: no CUDA
compute call is made here."""
import ctypes
import os
import re

import numpy as np
import pytest

import bj_synth as S
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_icpp_anztdfq17_b200", "libbj.so")


def _declared():
    names = set()
    for h in ("bj.h", "bj_synth.h"):
        txt = open(os.path.join(ROOT, "include", h)).read()
        txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
        for m in re.finditer(r"^\s*(?:const\s+char\s*\*|bj_status|int64_t|void|size_t)\s*\**\s*(bj_\w+)\s*\(",
                             txt, flags=re.M):
            names.add(m.group(1))
    return names


@pytest.fixture(scope="module")
def lib():
    if not os.path.exists(LIB):
        from paper_conf_icpp_anztdfq17_b200 import build
        build.build()
    return ctypes.CDLL(LIB)


def test_every_declared_symbol_is_exported(lib):
    names = _declared()
    assert len(names) >= 20
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    from paper_conf_icpp_anztdfq17_b200 import bj
    assert set(bj.EXPORTS) == names


def test_library_is_sm100a_only():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", LIB], capture_output=True, text=True).stdout
    arches = set(re.findall(r"sm_(\d+a?)", out))
    assert arches == {"100a"}, arches


def test_status_strings_and_version(lib):
    lib.bj_status_string.restype = ctypes.c_char_p
    lib.bj_status_string.argtypes = [ctypes.c_int]
    assert lib.bj_status_string(0) == b"BJ_OK"
    assert b"ALIGN" in lib.bj_status_string(-3)
    lib.bj_version.restype = ctypes.c_char_p
    assert b"sm_100a" in lib.bj_version()


def test_partition_matches_oracle():
    from paper_conf_icpp_anztdfq17_b200 import bj
    rng = np.random.default_rng(31)
    for _ in range(200):
        nb = int(rng.integers(0, 60))
        G = int(rng.integers(1, 9))
        sizes = rng.integers(0, 33, size=nb).astype(np.int32)
        assert bj.partition(sizes, G).tolist() == oracle.partition(sizes, G).tolist()
    sizes = S.block_sizes(1_000_000, 4, 32)
    for G in (1, 2, 4, 8):
        assert np.array_equal(bj.partition(sizes, G), oracle.partition(sizes, G))


def test_errors_without_gpu_are_arguments(lib):
    """Argument checks run before any CUDA call."""
    lib.bj_layout.argtypes = [ctypes.c_int64, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                              ctypes.c_void_p]
    assert lib.bj_layout(-1, None, 1, None, None, None) == -1
    assert lib.bj_layout(4, None, 7, None, None, None) == -1
    lib.bj_partition.argtypes = [ctypes.c_int64, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
    assert lib.bj_partition(3, None, 0, None) == -1
    lib.bj_supervariable_blocking.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p,
                                              ctypes.c_void_p]
    assert lib.bj_supervariable_blocking(None, 8, None, None, None) == -1
    csr = (ctypes.c_int64 * 8)(4, 0, 0, 0, 0, 0, 0, 0)          # nrows = 4, row_ptr = NULL
    nb = ctypes.c_int64(0)
    assert lib.bj_supervariable_blocking(ctypes.cast(csr, ctypes.c_void_p), 33, ctypes.c_void_p(16), ctypes.byref(nb),
                                         None) == -1


def test_gesv_host_rejects_short_buffers():
    """bj_gesv_host checks nvalues / nvec against the layout of sizes_h on the
    host, before any device work (so this runs without a GPU)."""
    from paper_conf_icpp_anztdfq17_b200 import bj
    L = bj.lib()
    ws = ctypes.c_void_p()
    assert L.bj_workspace_create(ctypes.byref(ws)) == 0
    sizes = np.array([3, 32, 1, 0, 7], dtype=np.int32)
    vec, val = oracle.layout(sizes, 8)
    need_val, need_vec = int(val[-1]), int(vec[-1])
    A = np.zeros(need_val, np.float64)
    b = np.zeros(need_vec, np.float64)
    x = np.zeros(need_vec, np.float64)
    P = lambda a: a.ctypes.data_as(ctypes.c_void_p)
    for nvalues, nvec in ((need_val - 1, need_vec), (need_val, need_vec - 1), (0, 0)):
        st = L.bj_gesv_host(ws, len(sizes), P(sizes), nvalues, P(A), nvec, P(b), P(x), None, None, 1, None)
        assert st == -1, (nvalues, nvec, st)
    L.bj_workspace_destroy(ws)
