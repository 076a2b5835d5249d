"""ctypes binding of libvegen.so -- the seeded synthetic-input generator.

Test / bench INPUTS ONLY (no analysis arithmetic).  Both the oracle-side
tests and the CUDA path use it; see include/ve_gen.h and DESIGN.md section 4.
"""
import ctypes
import os

import numpy as np

CFG1, CFG2, CFG3, CFG4, CFG5, FUZZ = 1, 2, 3, 4, 5, 100
SEEDS = {CFG1: 1, CFG2: 2, CFG3: 3, CFG4: 4, CFG5: 5}


def scaled(cfg, shift):
    """cfg code of cfg3 / cfg4 / cfg5 with every tensor 2^shift times smaller (0 = full size)."""
    return cfg | (shift << 8)

REC_DTYPE = np.dtype([("addr", "<u8"), ("value", "<u8"), ("pc", "<u4"), ("meta", "<u4")])
assert REC_DTYPE.itemsize == 24

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None


class VegRecord(ctypes.Structure):
    _fields_ = [("addr", ctypes.c_uint64), ("value", ctypes.c_uint64), ("pc", ctypes.c_uint32),
                ("meta", ctypes.c_uint32)]


class VegObject(ctypes.Structure):
    _fields_ = [("base", ctypes.c_uint64), ("size", ctypes.c_uint64), ("id", ctypes.c_uint32),
                ("elem_width", ctypes.c_uint32), ("has_pre", ctypes.c_uint32), ("has_post", ctypes.c_uint32)]


class VegInfo(ctypes.Structure):
    _fields_ = [("n_records", ctypes.c_uint64), ("n_pcs", ctypes.c_uint32), ("n_obj", ctypes.c_uint32),
                ("n_epochs", ctypes.c_uint32), ("pad", ctypes.c_uint32)]


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libvegen.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(path)
        u64, u32, i32, vp = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int, ctypes.c_void_p
        L.veg_info_get.argtypes = [i32, i32, ctypes.POINTER(VegInfo)]
        L.veg_object_get.argtypes = [i32, i32, u32, ctypes.POINTER(VegObject)]
        L.veg_records_host.argtypes = [i32, i32, u64, u64, u64, vp]
        L.veg_records_host.restype = None
        L.veg_records_device.argtypes = [i32, i32, u64, u64, u64, vp, vp]
        L.veg_snapshot_host.argtypes = [i32, i32, u64, u32, i32, u64, u64, vp]
        L.veg_snapshot_host.restype = None
        L.veg_snapshot_device.argtypes = [i32, i32, u64, u32, i32, vp, vp]
        L.veg_dedup_object.argtypes = [u64, u32, u64, ctypes.POINTER(VegObject), ctypes.POINTER(u32),
                                       ctypes.POINTER(u32)]
        L.veg_dedup_host.argtypes = [u64, u32, u64, vp]
        L.veg_dedup_host.restype = None
        L.veg_dedup_device.argtypes = [u64, u32, u64, vp, vp]
        _LIB = L
    return _LIB


def info(cfg, epoch=0):
    inf = VegInfo()
    if lib().veg_info_get(cfg, epoch, ctypes.byref(inf)) != 0:
        raise ValueError((cfg, epoch))
    return {"n_records": inf.n_records, "n_pcs": inf.n_pcs, "n_obj": inf.n_obj, "n_epochs": inf.n_epochs}


def objects(cfg, epoch=0):
    out = []
    for i in range(info(cfg, epoch)["n_obj"]):
        o = VegObject()
        if lib().veg_object_get(cfg, epoch, i, ctypes.byref(o)) != 0:
            raise ValueError(i)
        out.append({"base": o.base, "size": o.size, "id": o.id, "elem_width": o.elem_width,
                    "has_pre": bool(o.has_pre), "has_post": bool(o.has_post)})
    return out


def records_host(cfg, epoch, seed, r0, n):
    a = np.empty(n, dtype=REC_DTYPE)
    if n:
        lib().veg_records_host(cfg, epoch, seed, r0, n, a.ctypes.data)
    return a


def snapshot_host(cfg, epoch, seed, obj, post, off=0, length=None):
    if length is None:
        length = objects(cfg, epoch)[obj]["size"] - off
    a = np.empty(length, dtype=np.uint8)
    lib().veg_snapshot_host(cfg, epoch, seed, obj, int(post), off, length, a.ctypes.data)
    return a


def records_device(cfg, epoch, seed, r0, n, d_ptr, stream_ptr=0):
    if lib().veg_records_device(cfg, epoch, seed, r0, n, ctypes.c_void_p(d_ptr), ctypes.c_void_p(stream_ptr)) != 0:
        raise RuntimeError("veg_records_device failed")


def snapshot_device(cfg, epoch, seed, obj, post, d_ptr, stream_ptr=0):
    if lib().veg_snapshot_device(cfg, epoch, seed, obj, int(post), ctypes.c_void_p(d_ptr),
                                 ctypes.c_void_p(stream_ptr)) != 0:
        raise RuntimeError("veg_snapshot_device failed")


def dedup_object(seed, i, unit):
    o = VegObject()
    cls, src = ctypes.c_uint32(), ctypes.c_uint32()
    if lib().veg_dedup_object(seed, i, unit, ctypes.byref(o), ctypes.byref(cls), ctypes.byref(src)) != 0:
        raise ValueError(i)
    return {"base": o.base, "size": o.size, "id": o.id, "elem_width": o.elem_width, "cls": cls.value,
            "src": src.value}


def dedup_host(seed, i, unit):
    size = dedup_object(seed, i, unit)["size"]
    a = np.empty(size, dtype=np.uint8)
    lib().veg_dedup_host(seed, i, unit, a.ctypes.data)
    return a


def dedup_device(seed, i, unit, d_ptr, stream_ptr=0):
    if lib().veg_dedup_device(seed, i, unit, ctypes.c_void_p(d_ptr), ctypes.c_void_p(stream_ptr)) != 0:
        raise RuntimeError("veg_dedup_device failed")


_M64 = (1 << 64) - 1


def _mix64(z):
    z = (z + 0x9E3779B97F4A7C15) & _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def _h(seed, stream, i):
    return _mix64((_mix64(seed ^ ((stream * 0xD1B54A32D192ED03) & _M64)) + i) & _M64)


def c5_role(k, p):
    """cfg1 role of PC p of cfg5 kernel k (ve_gen_core.h veg_c5_role, geometry seed 5)"""
    return _h(5, 502, k * 64 + p) % 16
