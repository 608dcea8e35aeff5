"""CPU oracle of the GPU-FPX exception scan — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product (``paper_conf_hpdc_lilfslg23_b200``) never does.

This is a thin ctypes wrapper over ``fpx_oracle.cpp`` (plain single-threaded
C++17; see its header for what it computes and which paper passages each
function follows).  It shares no code with the CUDA path.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liborcfpx.so")

ENTRY_DTYPE = np.dtype(
    [
        ("site", "<u4"),
        ("kind", "u1"),
        ("flow", "u1"),
        ("fmt", "u1"),
        ("detail", "u1"),
        ("count", "<u8"),
        ("first_index", "<u8"),
    ]
)
assert ENTRY_DTYPE.itemsize == 24

CLEAN, C_NAN, C_INF, C_SUB = 0, 1, 2, 3

_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `python __graft_entry__.py build` first")
        L = ctypes.CDLL(_LIB_PATH)
        vp, u64, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
        L.orc_new.restype = vp
        L.orc_free.argtypes = [vp]
        L.orc_clear.argtypes = [vp]
        L.orc_classify.argtypes = [u32, u64]
        L.orc_classify.restype = ctypes.c_int
        L.orc_class_hist_fp32.argtypes = [u32, u32, vp]
        L.orc_dest_kind.argtypes = [u32, u32, u64, vp, u32]
        L.orc_dest_kind.restype = ctypes.c_int
        L.orc_scan_records.argtypes = [vp, vp, u64, vp, u64, u64, u32]
        L.orc_scan_tensor.argtypes = [vp, vp, u64, u32, u32, u64]
        L.orc_size.argtypes = [vp]
        L.orc_size.restype = u64
        L.orc_bad_records.argtypes = [vp]
        L.orc_bad_records.restype = u64
        L.orc_lane_values.argtypes = [vp]
        L.orc_lane_values.restype = u64
        L.orc_fetch.argtypes = [vp, vp, u64]
        L.orc_fetch.restype = u64
        L.orc_sizeof_hdr.restype = u32
        L.orc_sizeof_entry.restype = u32
        L.orc_key.argtypes = [u32, u32, u32, u32]
        L.orc_key.restype = u64
        assert L.orc_sizeof_hdr() == 16 and L.orc_sizeof_entry() == 24
        _lib = L
    return _lib


def classify(fmt: int, bits: int) -> int:
    return lib().orc_classify(fmt, bits)


def dest_kind(opclass: int, fmt: int, d: int, srcs=None) -> int:
    """Kind code (0 NaN, 1 INF, 2 SUB, 3 DIV0) of a destination value, -1 = none."""
    if srcs is None:
        return lib().orc_dest_kind(opclass, fmt, d, None, 0)
    a = np.asarray(srcs, dtype=np.uint64)
    return lib().orc_dest_kind(opclass, fmt, d, a.ctypes.data, len(a))


def class_hist_fp32(lo: int, hi: int) -> np.ndarray:
    c = np.zeros(4, dtype=np.uint64)
    lib().orc_class_hist_fp32(lo, hi, c.ctypes.data)
    return c


class Table:
    """The oracle's ordered exception table (std::map key -> count, first)."""

    def __init__(self):
        self._t = lib().orc_new()

    def __del__(self):
        if getattr(self, "_t", None):
            lib().orc_free(self._t)
            self._t = None

    def clear(self):
        lib().orc_clear(self._t)

    def scan_records(self, hdr: np.ndarray, arena: np.ndarray, base_index: int = 0, mode: int = 0):
        hdr = np.ascontiguousarray(hdr)
        arena = np.ascontiguousarray(arena)
        planes = arena.size // 32
        lib().orc_scan_records(self._t, hdr.ctypes.data, len(hdr), arena.ctypes.data, planes, base_index, mode)

    def scan_tensor(self, buf: np.ndarray, fmt: int, site: int, base_index: int = 0):
        buf = np.ascontiguousarray(buf)
        esize = {0: 4, 1: 8, 2: 2, 3: 2}[fmt]
        n = buf.nbytes // esize
        lib().orc_scan_tensor(self._t, buf.ctypes.data, n, fmt, site, base_index)

    @property
    def bad_records(self) -> int:
        return lib().orc_bad_records(self._t)

    @property
    def lane_values(self) -> int:
        return lib().orc_lane_values(self._t)

    def __len__(self):
        return lib().orc_size(self._t)

    def entries(self) -> np.ndarray:
        n = len(self)
        out = np.zeros(max(n, 1), dtype=ENTRY_DTYPE)
        got = lib().orc_fetch(self._t, out.ctypes.data, n)
        return out[:got]


def key(site: int, fmt: int, flow: int, kind: int) -> int:
    return lib().orc_key(site, fmt, flow, kind)
