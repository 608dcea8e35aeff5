"""fpxgen — seeded, counter-based synthetic inputs for the GPU-FPX scan.

Shared by both sides of the parity check (the oracle in ``oracle/`` and the
CUDA path in ``paper_conf_hpdc_lilfslg23_b200``) and by ``bench.py``.  It holds
none of the method's arithmetic: it never classifies a value, it only builds
clean values inside the normal range and writes planted exceptional bit
patterns (see ``csrc/gen_core.h`` for the recipe).

Host generation returns numpy arrays; device generation returns torch tensors
(int32 storage holding the raw 32-bit words).
"""
from __future__ import annotations

import ctypes
import dataclasses
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libfpxgen.so")

RECIPE_C1, RECIPE_MIX, RECIPE_FLOW, RECIPE_PACKED, RECIPE_STRESS = range(5)

HDR_DTYPE = np.dtype([("site", "<u4"), ("active_mask", "<u4"), ("meta", "<u4"), ("val_off", "<u4")])
WRITE_DTYPE = np.dtype(
    [("record", "<u8"), ("plane", "<u4"), ("lanemask", "<u4"), ("and_mask", "<u4"), ("or_bits", "<u4")]
)
INJ_DTYPE = np.dtype(
    [
        ("record", "<u8"),
        ("lanemask", "<u4"),
        ("dest_class", "u1"),
        ("src_class", "u1"),
        ("flow_intent", "u1"),
        ("slot", "u1"),
    ]
)
assert HDR_DTYPE.itemsize == 16 and WRITE_DTYPE.itemsize == 24 and INJ_DTYPE.itemsize == 16


class _Params(ctypes.Structure):
    _fields_ = [
        ("seed", ctypes.c_uint64),
        ("n_records", ctypes.c_uint64),
        ("n_sites", ctypes.c_uint32),
        ("recipe", ctypes.c_uint32),
        ("p_fp64_ppm", ctypes.c_uint32),
        ("p_partial_ppm", ctypes.c_uint32),
        ("p_zero_ppm", ctypes.c_uint32),
        ("dense_nan_ppm", ctypes.c_uint32),
    ]


@dataclasses.dataclass
class Params:
    """One synthetic trace.  ``n_records`` is the chunk length; records are
    numbered globally from ``r0`` (passed to the generate calls)."""

    seed: int
    n_records: int
    n_sites: int
    recipe: int = RECIPE_MIX
    p_fp64: float = 0.5
    p_partial: float = 0.10
    p_zero: float = 0.01
    dense_nan: float = 0.0
    zipf_s: float = 1.1

    def c(self) -> _Params:
        return _Params(
            self.seed,
            self.n_records,
            self.n_sites,
            self.recipe,
            int(round(self.p_fp64 * 1e6)),
            int(round(self.p_partial * 1e6)),
            int(round(self.p_zero * 1e6)),
            int(round(self.dense_nan * 1e6)),
        )


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run `python __graft_entry__.py build` first")
        L = ctypes.CDLL(_LIB_PATH)
        P = ctypes.POINTER(_Params)
        vp, u64, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
        L.fpxgen_zipf_cdf.argtypes = [u32, ctypes.c_double, vp]
        L.fpxgen_zipf_cdf.restype = None
        L.fpxgen_headers_host.argtypes = [P, vp, u64, u64, vp]
        L.fpxgen_headers_host.restype = u64
        L.fpxgen_fill_host.argtypes = [P, u64, vp, u64, vp]
        L.fpxgen_fill_host.restype = None
        L.fpxgen_plan_injections.argtypes = [P, vp, u64, u64, u32, u32, vp, u64, vp, u64, ctypes.POINTER(u64)]
        L.fpxgen_plan_injections.restype = ctypes.c_int64
        L.fpxgen_apply_host.argtypes = [vp, u64, vp, vp]
        L.fpxgen_apply_host.restype = None
        L.fpxgen_headers_device.argtypes = [P, vp, u64, u64, vp, ctypes.POINTER(u64), vp]
        L.fpxgen_headers_device.restype = ctypes.c_int
        L.fpxgen_fill_device.argtypes = [P, u64, vp, u64, vp, vp]
        L.fpxgen_fill_device.restype = ctypes.c_int
        L.fpxgen_apply_device.argtypes = [vp, u64, vp, vp, vp]
        L.fpxgen_apply_device.restype = ctypes.c_int
        L.fpxgen_last_error.restype = ctypes.c_char_p
        for f in ("fpxgen_sizeof_hdr", "fpxgen_sizeof_write", "fpxgen_sizeof_injection"):
            getattr(L, f).restype = u32
        assert L.fpxgen_sizeof_hdr() == 16 and L.fpxgen_sizeof_write() == 24
        assert L.fpxgen_sizeof_injection() == INJ_DTYPE.itemsize
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def zipf_cdf(n_sites: int, s: float) -> np.ndarray:
    cdf = np.empty(n_sites, dtype=np.float64)
    lib().fpxgen_zipf_cdf(n_sites, s, _ptr(cdf))
    return cdf


def generate_host(p: Params, r0: int = 0):
    """Headers (structured HDR_DTYPE array) and arena (uint32 [planes, 32])."""
    L = lib()
    cp = p.c()
    cdf = zipf_cdf(p.n_sites, p.zipf_s)
    hdr = np.empty(p.n_records, dtype=HDR_DTYPE)
    planes = L.fpxgen_headers_host(ctypes.byref(cp), _ptr(cdf), r0, p.n_records, _ptr(hdr))
    arena = np.zeros((max(planes, 1), 32), dtype=np.uint32)
    L.fpxgen_fill_host(ctypes.byref(cp), r0, _ptr(hdr), p.n_records, _ptr(arena))
    return hdr, arena[:planes] if planes else arena[:0]


def plan_injections(p: Params, n_inj: int, storm_frac: float = 0.2, flow: bool = False, r0: int = 0):
    """Planted events (INJ_DTYPE, record numbers chunk-relative) and writes."""
    L = lib()
    cp = p.c()
    cdf = zipf_cdf(p.n_sites, p.zipf_s)
    nw = ctypes.c_uint64(0)
    storm_ppm = int(round(storm_frac * 1e6))
    ni = L.fpxgen_plan_injections(ctypes.byref(cp), _ptr(cdf), r0, n_inj, storm_ppm, int(flow), None, 0, None, 0,
                                  ctypes.byref(nw))
    inj = np.zeros(max(ni, 1), dtype=INJ_DTYPE)
    wr = np.zeros(max(nw.value, 1), dtype=WRITE_DTYPE)
    nw2 = ctypes.c_uint64(0)
    ni2 = L.fpxgen_plan_injections(ctypes.byref(cp), _ptr(cdf), r0, n_inj, storm_ppm, int(flow), _ptr(inj), ni,
                                   _ptr(wr), nw.value, ctypes.byref(nw2))
    assert ni2 == ni and nw2.value == nw.value
    return inj[:ni], wr[: nw.value]


def apply_host(writes: np.ndarray, hdr: np.ndarray, arena: np.ndarray) -> None:
    if len(writes):
        lib().fpxgen_apply_host(_ptr(writes), len(writes), _ptr(hdr), _ptr(arena))


def generate_device(p: Params, r0: int = 0, device=None, stream=None):
    """Same bytes as generate_host, built in HBM.  Returns (hdr int32 [n,4],
    arena int32 [planes*32], planes)."""
    import torch

    L = lib()
    cp = p.c()
    dev = torch.device("cuda", torch.cuda.current_device() if device is None else device)
    cdf = torch.from_numpy(zipf_cdf(p.n_sites, p.zipf_s)).to(dev)
    hdr = torch.empty((max(p.n_records, 1), 4), dtype=torch.int32, device=dev)
    s = torch.cuda.current_stream(dev) if stream is None else stream
    planes = ctypes.c_uint64(0)
    rc = L.fpxgen_headers_device(ctypes.byref(cp), cdf.data_ptr(), r0, p.n_records, hdr.data_ptr(),
                                 ctypes.byref(planes), s.cuda_stream)
    if rc != 0:
        raise RuntimeError(f"fpxgen_headers_device: {L.fpxgen_last_error().decode()}")
    arena = torch.empty(max(planes.value, 1) * 32, dtype=torch.int32, device=dev)
    rc = L.fpxgen_fill_device(ctypes.byref(cp), r0, hdr.data_ptr(), p.n_records, arena.data_ptr(), s.cuda_stream)
    if rc != 0:
        raise RuntimeError(f"fpxgen_fill_device: {L.fpxgen_last_error().decode()}")
    return hdr[: p.n_records], arena, planes.value


def apply_device(writes: np.ndarray, hdr, arena, stream=None) -> None:
    import torch

    if len(writes) == 0:
        return
    L = lib()
    w = torch.from_numpy(writes.view(np.uint8).copy()).to(hdr.device)
    s = torch.cuda.current_stream(hdr.device) if stream is None else stream
    rc = L.fpxgen_apply_device(w.data_ptr(), len(writes), hdr.data_ptr(), arena.data_ptr(), s.cuda_stream)
    if rc != 0:
        raise RuntimeError(f"fpxgen_apply_device: {L.fpxgen_last_error().decode()}")
    s.synchronize()  # keep `w` alive until the kernel has run
