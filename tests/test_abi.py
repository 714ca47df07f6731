"""CPU checks of the boundary: librtm.so loads and exports every symbol include/rtm.h declares;
layouts agree with the header; the product package never imports the oracle."""
from __future__ import annotations

import ctypes
import os
import re
import subprocess

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "rtm.h")
PKG = os.path.join(ROOT, "paper_conf_micro_mosallaeii024_b200")


def _declared():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(rtm_[a-z_]+)\s*\(", text)) - {"rtm_allgather_fn"})


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(os.path.join(PKG, "librtm.so"))
    names = _declared()
    assert len(names) >= 15
    for n in names:
        assert hasattr(lib, n), n
    from paper_conf_micro_mosallaeii024_b200 import _native

    assert set(_native.EXPORTS) == set(names)


def test_library_is_built_for_sm100a():
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", os.path.join(PKG, "librtm.so")],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings_and_version():
    from paper_conf_micro_mosallaeii024_b200 import _native as N

    L = N.lib()
    for code in (0, -1, -2, -3, -4, -5, -6, -7):
        assert L.rtm_status_str(code)
    assert b"sm_100a" in L.rtm_version()


def test_create_rejects_bad_config_without_gpu_work():
    """Argument validation happens before any device call (returns RTM_E_INVALID)."""
    from paper_conf_micro_mosallaeii024_b200 import _native as N

    L = N.lib()
    owner = np.zeros(4, np.uint32)
    cap = np.array([4, 8, 0, 4], np.uint16)  # capacity 0 is invalid
    tot = np.ones(1, np.int64)
    cfg = N.Config()
    cfg.n_buffers, cfg.n_components, cfg.n_kernels = 4, 1, 1
    cfg.buffer_owner, cfg.buffer_capacity, cfg.kernel_total = owner.ctypes.data, cap.ctypes.data, tot.ctypes.data
    cfg.hang_windows, cfg.k, cfg.world = 1, 4, 1
    h = ctypes.c_void_p()
    assert L.rtm_create(ctypes.byref(cfg), ctypes.byref(h)) == N.RTM_E_INVALID
    cap[2] = 65535  # reserved value
    assert L.rtm_create(ctypes.byref(cfg), ctypes.byref(h)) == N.RTM_E_INVALID
    cap[2] = 8
    cfg.k = 0
    assert L.rtm_create(ctypes.byref(cfg), ctypes.byref(h)) == N.RTM_E_INVALID
    assert L.rtm_window_reduce(None, None, 0, None) == N.RTM_E_INVALID


def test_record_and_result_layouts_match_header():
    from paper_conf_micro_mosallaeii024_b200 import _native as N

    assert N.SAMPLE_DTYPE.itemsize == 16 and N.EVENT_DTYPE.itemsize == 16
    assert N.SUMMARY_DTYPE.itemsize == 56 and N.BSTAT_DTYPE.itemsize == 32
    assert N.TOPK_DTYPE.itemsize == 8 and N.PROGRESS_DTYPE.itemsize == 40 and N.COMP_DTYPE.itemsize == 24
    import gen

    assert N.SAMPLE_DTYPE == gen.SAMPLE_DTYPE and N.EVENT_DTYPE == gen.EVENT_DTYPE


def test_product_never_touches_the_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "liboracle" not in src and "oracle.h" not in src, f


def test_kernel_launch_counter_is_monotone_without_gpu():
    """rtm_kernel_launches needs no device: it only reads the library's launch counter."""
    from paper_conf_micro_mosallaeii024_b200 import _native

    L = _native.lib()
    a = L.rtm_kernel_launches()
    b = L.rtm_kernel_launches()
    assert b >= a >= 0
