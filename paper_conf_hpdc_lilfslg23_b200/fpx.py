"""Thin ctypes binding of libfpx.so (include/fpx.h): argument marshalling only.

Every step of the scan runs in the library's sm_100a kernels; this module
passes device pointers (torch tensors) and the current CUDA stream.  It never
falls back to the CPU: if ``libfpx.so`` is missing the import fails.

Low-level names mirror the C ABI (``fpx_open``, ``fpx_scan_records``, ...);
``Handle`` is a small convenience wrapper used by tests, bench and ``dist``.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.environ.get("FPX_LIB") or os.path.join(_HERE, "libfpx.so")  # FPX_LIB: A/B builds (tuning)
if not os.path.exists(_LIB_PATH):
    raise ImportError(f"{_LIB_PATH} is missing: build it with `python __graft_entry__.py build` (no CPU fallback)")
lib = ctypes.CDLL(_LIB_PATH)

# ---- enums (include/fpx.h) ---------------------------------------------------
OK, ERR_INVALID, ERR_CUDA, ERR_NOMEM, ERR_TABLE_FULL, ERR_BAD_RECORD, ERR_TRUNCATED = 0, -1, -2, -3, -4, -5, -6
FP32, FP64, FP16, BF16 = 0, 1, 2, 3
NAN, INF, SUB, DIV0 = 0, 1, 2, 3
FLOW_NONE, GEN, PROP, KILL = 0, 1, 2, 3
MODE_DEST, MODE_FLOW, MODE_FLOW_DETAIL = 0, 1, 2
DETAIL_CMP = 4
FETCH_ALL, FETCH_NEW = 0, 1
OPT_SCAN_LDG = 1
OPT_NO_WARP_AGG = 2  # ablation: no warp aggregation in the record scans' exact path
OPT_LIVE_NEW = 4  # early notification: new keys published to mapped host memory (fpx_poll_new)
OPT_STORM = 8  # always the record scan's storm kernel (else chosen from the previous scan's density)
KEY_EMPTY = 0xFFFFFFFFFFFFFFFF

ENTRY_DTYPE = np.dtype(
    [("site", "<u4"), ("kind", "u1"), ("flow", "u1"), ("fmt", "u1"), ("detail", "u1"), ("count", "<u8"),
     ("first_index", "<u8")]
)
HDR_DTYPE = np.dtype([("site", "<u4"), ("active_mask", "<u4"), ("meta", "<u4"), ("val_off", "<u4")])


class IpcTable(ctypes.Structure):
    _fields_ = [("ipc", (ctypes.c_ubyte * 64) * 4), ("table_log2_slots", ctypes.c_uint32),
                ("newlog_capacity", ctypes.c_uint32), ("home_device", ctypes.c_int32), ("magic", ctypes.c_uint32)]


class TensorDesc(ctypes.Structure):
    _fields_ = [("ptr", ctypes.c_void_p), ("n_elems", ctypes.c_uint64), ("base_index", ctypes.c_uint64),
                ("fmt", ctypes.c_uint32), ("site", ctypes.c_uint32)]


class Options(ctypes.Structure):
    _fields_ = [("table_log2_slots", ctypes.c_uint32), ("newlog_capacity", ctypes.c_uint32),
                ("flags", ctypes.c_uint32)]


class Stats(ctypes.Structure):
    _fields_ = [("bad_records", ctypes.c_uint64), ("dropped_events", ctypes.c_uint64),
                ("table_entries", ctypes.c_uint64), ("newlog_overflow", ctypes.c_uint64)]


_vp, _u64, _u32, _st = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
_P64 = ctypes.POINTER(ctypes.c_uint64)
_SIGS = {
    "fpx_open": ([ctypes.c_int, ctypes.POINTER(Options), ctypes.POINTER(_vp)], _st),
    "fpx_scan_records": ([_vp, _vp, _u64, _vp, _u64, _u64, _u32, _vp], _st),
    "fpx_scan_tensor": ([_vp, _vp, _u64, _u32, _u32, _u64, _vp], _st),
    "fpx_scan_tensors": ([_vp, ctypes.POINTER(TensorDesc), _u32, _vp], _st),
    "fpx_table_fetch": ([_vp, _vp, _u64, _P64, _u32], _st),
    "fpx_table_fetch_device": ([_vp, _vp, _vp, _vp, _u64, _P64, _vp], _st),
    "fpx_table_lookup_device": ([_vp, _vp, _u64, _vp, _vp, _vp], _st),
    "fpx_keys_unique_device": ([_vp, _vp, _u64, _vp, _P64, _vp], _st),
    "fpx_table_merge_device": ([_vp, _vp, _vp, _vp, _u64, _vp], _st),
    "fpx_table_reset": ([_vp, _vp], _st),
    "fpx_get_stats": ([_vp, ctypes.POINTER(Stats)], _st),
    "fpx_poll_new": ([_vp, _vp, _u64, _P64], _st),
    "fpx_table_export": ([_vp, ctypes.POINTER(IpcTable)], _st),
    "fpx_open_attached": ([ctypes.c_int, ctypes.POINTER(IpcTable), ctypes.POINTER(_vp)], _st),
    "fpx_close": ([_vp], _st),
    "fpx_strerror": ([_st], ctypes.c_char_p),
    "fpx_last_cuda_error": ([], ctypes.c_char_p),
    "fpx_abi_version": ([], _u32),
    "fpx_sizeof_rec_hdr": ([], _u32),
    "fpx_sizeof_entry": ([], _u32),
}
EXPORTS = tuple(_SIGS)
for _name, (_args, _res) in _SIGS.items():
    if os.environ.get("FPX_LIB") and not hasattr(lib, _name):  # A/B against an older build (tuning only)
        continue
    _f = getattr(lib, _name)
    _f.argtypes = _args
    _f.restype = _res
    globals()[_name] = _f
assert lib.fpx_sizeof_rec_hdr() == 16 and lib.fpx_sizeof_entry() == 24


class FpxError(RuntimeError):
    def __init__(self, status: int, where: str):
        msg = lib.fpx_strerror(status).decode()
        if status == ERR_CUDA:
            msg += f" ({lib.fpx_last_cuda_error().decode()})"
        super().__init__(f"{where}: {msg} [{status}]")
        self.status = status


def check(status: int, where: str, allow=()) -> int:
    if status != OK and status not in allow:
        raise FpxError(status, where)
    return status


def _stream_ptr(stream) -> int:
    import torch

    s = torch.cuda.current_stream() if stream is None else stream
    return s.cuda_stream


class Handle:
    """One fpx context on one device (fpx_open ... fpx_close)."""

    def __init__(self, device: int = 0, table_log2_slots: int = 0, newlog_capacity: int = 0, flags: int = 0):
        self._h = _vp()
        opt = Options(table_log2_slots, newlog_capacity, flags)
        check(lib.fpx_open(device, ctypes.byref(opt), ctypes.byref(self._h)), "fpx_open")
        self.device = device
        self.last_status = OK

    # context manager
    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def close(self):
        if self._h:
            check(lib.fpx_close(self._h), "fpx_close")
            self._h = _vp()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def ptr(self):
        return self._h

    def export(self) -> bytes:
        """The table as CUDA IPC handles (fpx_table_export), for attach()."""
        t = IpcTable()
        check(lib.fpx_table_export(self._h, ctypes.byref(t)), "fpx_table_export")
        return bytes(t)

    @classmethod
    def attach(cls, device: int, exported: bytes) -> "Handle":
        """A handle on `device` (in another process) whose scans update the
        exported table in place through peer memory (fpx_open_attached)."""
        self = cls.__new__(cls)
        self._h = _vp()
        t = IpcTable.from_buffer_copy(exported)
        check(lib.fpx_open_attached(device, ctypes.byref(t), ctypes.byref(self._h)), "fpx_open_attached")
        self.device = device
        self.last_status = OK
        return self

    def scan_records(self, hdr, arena, base_index: int = 0, mode: int = MODE_DEST, stream=None, n_records=None,
                     arena_planes=None):
        """hdr: device tensor of 16-B headers (e.g. int32 [n, 4]); arena: device
        tensor of 128-B planes (any dtype, contiguous)."""
        n = hdr.numel() * hdr.element_size() // 16 if n_records is None else n_records
        planes = arena.numel() * arena.element_size() // 128 if arena_planes is None else arena_planes
        check(lib.fpx_scan_records(self._h, hdr.data_ptr(), n, arena.data_ptr(), planes, base_index, mode,
                                   _stream_ptr(stream)), "fpx_scan_records")

    def scan_tensor(self, t, fmt: int | None = None, site: int = 0, base_index: int = 0, stream=None):
        import torch

        if fmt is None:
            fmt = {torch.float32: FP32, torch.float64: FP64, torch.float16: FP16, torch.bfloat16: BF16}[t.dtype]
        es = {FP32: 4, FP64: 8, FP16: 2, BF16: 2}[fmt]
        assert t.is_contiguous()
        n = t.numel() * t.element_size() // es
        check(lib.fpx_scan_tensor(self._h, t.data_ptr(), n, fmt, site, base_index, _stream_ptr(stream)),
              "fpx_scan_tensor")

    def scan_tensors(self, items, stream=None):
        """One launch for many tensors: items = [(tensor, site, base_index), ...]
        (fmt from the dtype).  fpx_scan_tensors."""
        import torch

        fmts = {torch.float32: FP32, torch.float64: FP64, torch.float16: FP16, torch.bfloat16: BF16}
        arr = (TensorDesc * max(len(items), 1))()
        for i, (t, site, base) in enumerate(items):
            assert t.is_contiguous()
            arr[i] = TensorDesc(t.data_ptr(), t.numel(), base, fmts[t.dtype], site)
        check(lib.fpx_scan_tensors(self._h, arr, len(items), _stream_ptr(stream)), "fpx_scan_tensors")

    def fetch(self, flags: int = FETCH_ALL, capacity: int | None = None) -> np.ndarray:
        """Entries ascending by key.  Sticky device statuses (bad record, table
        full) are kept in self.last_status, not raised."""
        if flags != FETCH_ALL:
            raise ValueError("use Handle.fetch_new() for FPX_FETCH_NEW")
        n = ctypes.c_uint64(0)
        check(lib.fpx_table_fetch(self._h, None, 0, ctypes.byref(n), flags), "fpx_table_fetch",
              allow=(ERR_TRUNCATED, ERR_BAD_RECORD, ERR_TABLE_FULL))
        cap = n.value if capacity is None else capacity
        out = np.zeros(max(cap, 1), dtype=ENTRY_DTYPE)
        st = check(lib.fpx_table_fetch(self._h, out.ctypes.data, cap, ctypes.byref(n), flags), "fpx_table_fetch",
                   allow=(ERR_TRUNCATED, ERR_BAD_RECORD, ERR_TABLE_FULL))
        self.last_status = st
        return out[: min(cap, n.value)]

    def fetch_new(self, capacity: int = 1 << 20) -> np.ndarray:
        """Keys first inserted since the previous fetch_new (FPX_FETCH_NEW), at
        most `capacity` of them in insertion order (sorted by key); a truncated
        call leaves the rest for the next one (last_status = ERR_TRUNCATED)."""
        n = ctypes.c_uint64(0)
        out = np.zeros(max(capacity, 1), dtype=ENTRY_DTYPE)
        st = check(lib.fpx_table_fetch(self._h, out.ctypes.data, capacity, ctypes.byref(n), FETCH_NEW),
                   "fpx_table_fetch", allow=(ERR_TRUNCATED, ERR_BAD_RECORD, ERR_TABLE_FULL))
        self.last_status = st
        return out[: min(capacity, n.value)]

    def poll_new(self, capacity: int = 4096) -> np.ndarray:
        """Keys inserted since the previous poll, while scans may still be
        running (fpx_poll_new; needs flags=OPT_LIVE_NEW).  count / first_index
        are the inserting event's (provisional)."""
        n = ctypes.c_uint64(0)
        out = np.zeros(max(capacity, 1), dtype=ENTRY_DTYPE)
        check(lib.fpx_poll_new(self._h, out.ctypes.data, capacity, ctypes.byref(n)), "fpx_poll_new")
        return out[: n.value]

    def fetch_device(self, capacity: int | None = None, stream=None):
        """(keys, counts, firsts) as int64 device tensors, sorted by key."""
        import torch

        dev = torch.device("cuda", self.device)
        n = ctypes.c_uint64(0)
        if capacity is None:
            capacity = int(self.stats().table_entries)  # exact upper bound, no extra fetch pass
        k = torch.empty(max(capacity, 1), dtype=torch.int64, device=dev)
        c = torch.empty_like(k)
        f = torch.empty_like(k)
        st = check(lib.fpx_table_fetch_device(self._h, k.data_ptr(), c.data_ptr(), f.data_ptr(), capacity,
                                              ctypes.byref(n), _stream_ptr(stream)),
                   "fpx_table_fetch_device", allow=(ERR_TRUNCATED, ERR_BAD_RECORD, ERR_TABLE_FULL))
        self.last_status = st
        m = min(capacity, n.value)
        return k[:m], c[:m], f[:m]

    def lookup_device(self, keys, stream=None):
        import torch

        c = torch.empty_like(keys)
        f = torch.empty_like(keys)
        check(lib.fpx_table_lookup_device(self._h, keys.data_ptr(), keys.numel(), c.data_ptr(), f.data_ptr(),
                                          _stream_ptr(stream)), "fpx_table_lookup_device")
        return c, f

    def unique_device(self, keys, stream=None):
        import torch

        out = torch.empty_like(keys)
        n = ctypes.c_uint64(0)
        check(lib.fpx_keys_unique_device(self._h, keys.data_ptr(), keys.numel(), out.data_ptr(), ctypes.byref(n),
                                         _stream_ptr(stream)), "fpx_keys_unique_device")
        return out[: n.value]

    def merge_device(self, keys, counts, firsts, stream=None):
        check(lib.fpx_table_merge_device(self._h, keys.data_ptr(), counts.data_ptr(), firsts.data_ptr(), keys.numel(),
                                         _stream_ptr(stream)), "fpx_table_merge_device")

    def reset(self, stream=None):
        check(lib.fpx_table_reset(self._h, _stream_ptr(stream)), "fpx_table_reset")

    def stats(self) -> Stats:
        s = Stats()
        check(lib.fpx_get_stats(self._h, ctypes.byref(s)), "fpx_get_stats")
        return s


def t4_summary(entries: np.ndarray) -> dict:
    """Table-4-style summary: number of distinct sites per
    (fmt, kind) over the fetched entries (any flow)."""
    out = {}
    for fmt in (FP32, FP64, FP16, BF16):
        for kind in (NAN, INF, SUB, DIV0):
            sel = entries[(entries["fmt"] == fmt) & (entries["kind"] == kind)]
            if len(sel):
                out[(fmt, kind)] = int(len(np.unique(sel["site"])))
    return out
