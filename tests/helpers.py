"""Small builders for hand-made traces (test inputs only; no analysis arithmetic)."""
import struct

import numpy as np

from gen.vegen import REC_DTYPE

U, S, F, BF = 0, 1, 2, 3          # kinds
LG = {1: 0, 2: 1, 4: 2, 8: 3}


def meta(w, kind, store=0, shared=0):
    return LG[w] | (kind << 2) | (store << 4) | (shared << 5)


def f32(x):
    return struct.unpack("<I", struct.pack("<f", x))[0]


def f64(x):
    return struct.unpack("<Q", struct.pack("<d", x))[0]


def as_f32(bits):
    return struct.unpack("<f", struct.pack("<I", bits))[0]


def records(rows):
    """rows: iterable of (addr, value, pc, meta)"""
    rows = list(rows)
    a = np.zeros(len(rows), dtype=REC_DTYPE)
    if rows:
        a["addr"] = np.array([int(r[0]) for r in rows], dtype=np.uint64)
        a["value"] = np.array([int(r[1]) for r in rows], dtype=np.uint64)
        a["pc"] = np.array([int(r[2]) for r in rows], dtype=np.uint32)
        a["meta"] = np.array([int(r[3]) for r in rows], dtype=np.uint32)
    return a


def obj(base, size, oid, ew, pre=None, post=None):
    return {"base": base, "size": size, "id": oid, "elem_width": ew, "pre": pre, "post": post}


def zeros(n):
    return np.zeros(n, dtype=np.uint8)


def le_bytes(values, w):
    """pack integer values little-endian, w bytes each"""
    out = bytearray()
    for v in values:
        out += int(v).to_bytes(w, "little")
    return np.frombuffer(bytes(out), dtype=np.uint8).copy()
