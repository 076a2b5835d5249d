"""ctypes harness of the CPU oracle (liboracle.so).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs -- never by the product
package.  See oracle/ve_oracle.h for what the oracle computes and where each
definition comes from.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

MAX_TOPK = 64
LINE_EMPTY, LINE_POINT, LINE_LINE, LINE_FAIL = 0, 1, 2, 3
DIFF_WRITTEN, DIFF_ALL, DIFF_MASK = 0, 1, 2
TYPE_NAMES = ["u8", "u16", "u32", "u64", "i8", "i16", "i32", "i64", "f16", "f32", "f64", "bf16"]

SUM_FIELDS = ["n_ld", "n_st", "n_zero", "n_ld_eq_pre", "n_st_eq_pre", "n_nosnap"]
FLAG_SUM_FIELDS = ["n_nan", "n_nonint", "n_not_f16", "n_not_bf16", "n_not_f32"]
MINMAX_FIELDS = ["raw_min", "raw_max", "ord_min", "ord_max", "trunc_min", "trunc_max"]
DERIVED_FIELDS = ["single_value", "single_zero", "frequent", "structured", "approx", "dict8", "heavy",
                  "single_type"]

KEY_DTYPE = np.dtype(
    [(f, "<u8") for f in SUM_FIELDS] + [("n_type", "<u8", (12,))] + [(f, "<u8") for f in FLAG_SUM_FIELDS]
    + [(f, "<u8") for f in MINMAX_FIELDS]
    + [("line_state", "<u8"), ("p_x", "<u8"), ("p_ylo", "<u8"), ("p_yhi", "<i8"), ("q_x", "<u8"),
       ("q_ylo", "<u8"), ("q_yhi", "<i8")]
    + [("n_distinct", "<u8"), ("n_top", "<u8"), ("top_bits", "<u8", (MAX_TOPK,)),
       ("top_count", "<u8", (MAX_TOPK,))]
    + [(f, "<u4") for f in DERIVED_FIELDS])
GLOB_DTYPE = np.dtype([("n_records", "<u8"), ("n_invalid", "<u8"), ("n_unmapped", "<u8"), ("u_touched", "<u8")])
OBJSTAT_DTYPE = np.dtype([("n_elems", "<u8"), ("n_written", "<u8"), ("n_loaded_eq", "<u8"),
                          ("n_ld_reload", "<u8"), ("n_touched", "<u8")])
INTERVAL_DTYPE = np.dtype([("start", "<u8"), ("end", "<u8")])
COPY_NONE, COPY_SEGMENT, COPY_MINMAX = 0, 1, 2
PLAN_DTYPE = np.dtype([(f, "<u8") for f in ("n_segments", "accessed_bytes", "lo", "hi", "direct_bytes",
                                           "minmax_bytes")] + [("choice", "<u4"), ("pad", "<u4")])
DIFF_DTYPE = np.dtype([("n_elems", "<u8"), ("n_masked", "<u8"), ("n_unchanged", "<u8"), ("n_changed", "<u8"),
                       ("n_untouched", "<u8"), ("redundant", "<u4"), ("pad", "<u4")])


class VoObject(ctypes.Structure):
    _fields_ = [("base", ctypes.c_uint64), ("size", ctypes.c_uint64), ("pre", ctypes.c_void_p),
                ("post", ctypes.c_void_p), ("id", ctypes.c_uint32), ("elem_width", ctypes.c_uint32)]


class VoConfig(ctypes.Structure):
    _fields_ = [("n_pcs", ctypes.c_uint32), ("topk", ctypes.c_uint32), ("mant_bits", ctypes.c_uint32),
                ("t_redundant_pct", ctypes.c_uint32), ("t_frequent_pct", ctypes.c_uint32),
                ("pad", ctypes.c_uint32)]


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build()")
        L = ctypes.CDLL(path)
        vp, u32, u64 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64
        L.vo_analyze.argtypes = [ctypes.POINTER(VoConfig), vp, u32, vp, u64, vp, vp, vp]
        L.vo_snapshot_diff.argtypes = [ctypes.POINTER(VoConfig), vp, u32, vp, u64, u32, u32, vp, vp]
        L.vo_object_dedup.argtypes = [vp, u32, vp]
        L.vo_vfg_build.argtypes = [vp, u64, vp, vp, vp, vp]
        L.vo_vfg_slice.argtypes = [vp, u64, vp, u64, u32, vp, vp, vp, vp]
        L.vo_vfg_important.argtypes = [vp, u64, vp, u64, u64, u64, vp, vp, vp, vp]
        L.vo_temporal_loads.argtypes = [ctypes.POINTER(VoConfig), vp, u32, vp, u64, vp]
        L.vo_approx_topk.argtypes = [ctypes.POINTER(VoConfig), vp, u32, vp, u64, vp, vp, vp]
        L.vo_interval_merge.argtypes = [vp, u64, vp]
        L.vo_interval_merge.restype = u64
        L.vo_record_intervals.argtypes = [u32, vp, u64, vp]
        L.vo_record_intervals.restype = u64
        L.vo_plan_copies.argtypes = [vp, u32, vp, u64, u32, u32, vp]
        L.vo_ord.argtypes = [u64, u32, u32]
        L.vo_ord.restype = u64
        L.vo_float_flags.argtypes = [u64, u32, u32]
        L.vo_float_flags.restype = u32
        L.vo_trunc.argtypes = [u64, u32, u32, u32]
        L.vo_trunc.restype = u64
        L.vo_sizeof.argtypes = [ctypes.c_int]
        L.vo_sizeof.restype = u64
        for which, dt in enumerate([KEY_DTYPE, GLOB_DTYPE, OBJSTAT_DTYPE, DIFF_DTYPE]):
            assert L.vo_sizeof(which) == dt.itemsize, (which, L.vo_sizeof(which), dt.itemsize)
        assert L.vo_sizeof(4) == ctypes.sizeof(VoObject)
        assert L.vo_sizeof(6) == PLAN_DTYPE.itemsize
        _LIB = L
    return _LIB


def make_config(n_pcs, topk=8, mant_bits=7, t_redundant_pct=33, t_frequent_pct=33):
    return VoConfig(n_pcs, topk, mant_bits, t_redundant_pct, t_frequent_pct, 0)


def _objects(objs):
    """objs: list of dicts {base, size, id, elem_width, pre (np.uint8 or None), post}."""
    arr = (VoObject * max(len(objs), 1))()
    keep = []
    for i, o in enumerate(objs):
        pre, post = o.get("pre"), o.get("post")
        for a in (pre, post):
            if a is not None:
                assert a.dtype == np.uint8 and a.flags.c_contiguous and len(a) >= o["size"]
                keep.append(a)
        arr[i] = VoObject(o["base"], o["size"], pre.ctypes.data if pre is not None else None,
                          post.ctypes.data if post is not None else None, o["id"], o["elem_width"])
    return arr, keep


def analyze(cfg, objs, recs):
    """Returns (keys[n_pcs + n_obj + 1], globals, objstat[n_obj]) as numpy structured arrays."""
    recs = np.ascontiguousarray(recs)
    assert recs.dtype.itemsize == 24
    arr, _keep = _objects(objs)
    n_keys = cfg.n_pcs + len(objs) + 1
    keys = np.zeros(n_keys, dtype=KEY_DTYPE)
    glob = np.zeros(1, dtype=GLOB_DTYPE)
    objstat = np.zeros(max(len(objs), 1), dtype=OBJSTAT_DTYPE)
    rc = lib().vo_analyze(ctypes.byref(cfg), arr, len(objs), recs.ctypes.data, len(recs), keys.ctypes.data,
                          glob.ctypes.data, objstat.ctypes.data)
    if rc != 0:
        raise ValueError("vo_analyze rejected its arguments")
    return keys, glob[0], objstat[:len(objs)]


def snapshot_diff(cfg, objs, recs, obj_id, mode=DIFF_WRITTEN, mask=None):
    recs = np.ascontiguousarray(recs)
    arr, _keep = _objects(objs)
    out = np.zeros(1, dtype=DIFF_DTYPE)
    m = None
    if mask is not None:
        m = np.ascontiguousarray(mask, dtype=np.uint32)
    rc = lib().vo_snapshot_diff(ctypes.byref(cfg), arr, len(objs), recs.ctypes.data, len(recs), obj_id, mode,
                                m.ctypes.data if m is not None else None, out.ctypes.data)
    if rc != 0:
        raise ValueError("vo_snapshot_diff rejected its arguments")
    return out[0]


def object_dedup(objs):
    arr, _keep = _objects(objs)
    g = np.zeros(max(len(objs), 1), dtype=np.uint32)
    lib().vo_object_dedup(arr, len(objs), g.ctypes.data)
    return g[:len(objs)]


def y_of(lo, hi):
    """signed 128-bit y of a line endpoint from its (lo, hi) halves"""
    return (int(hi) << 64) | int(lo)


def ord_key(b, kind, w):
    return lib().vo_ord(b, kind, w)


def float_flags(b, kind, w):
    return lib().vo_float_flags(b, kind, w)


def trunc(b, kind, w, K):
    return lib().vo_trunc(b, kind, w, K)


def interval_merge(intervals):
    """C13: intervals = INTERVAL_DTYPE array (or (n, 2) u64); returns the merged INTERVAL_DTYPE array."""
    iv = np.ascontiguousarray(np.asarray(intervals).view(np.uint64).reshape(-1, 2)).view(INTERVAL_DTYPE).ravel()
    out = np.zeros(max(len(iv), 1), dtype=INTERVAL_DTYPE)
    k = lib().vo_interval_merge(iv.ctypes.data, len(iv), out.ctypes.data)
    return out[:k]


def record_intervals(n_pcs, recs):
    """C14: merged intervals [addr, addr + w - 1] of the valid global-space records."""
    recs = np.ascontiguousarray(recs)
    out = np.zeros(max(len(recs), 1), dtype=INTERVAL_DTYPE)
    k = lib().vo_record_intervals(n_pcs, recs.ctypes.data, len(recs), out.ctypes.data)
    return out[:k]


def plan_copies(objs, merged, seg_max=32, dense_pct=50):
    """C15: per-object copy plan (PLAN_DTYPE indexed by object id)."""
    arr, _keep = _objects(objs)
    m = np.ascontiguousarray(merged, dtype=INTERVAL_DTYPE)
    out = np.zeros(max(len(objs), 1), dtype=PLAN_DTYPE)
    rc = lib().vo_plan_copies(arr, len(objs), m.ctypes.data, len(m), seg_max, dense_pct, out.ctypes.data)
    if rc != 0:
        raise ValueError("vo_plan_copies rejected its arguments")
    return out[:len(objs)]


def approx_topk(cfg, objs, recs):
    """C16: (ndistinct[n_keys], top_bits[n_keys, topk], top_count[n_keys, topk]) of the truncated values."""
    recs = np.ascontiguousarray(recs)
    arr, _keep = _objects(objs)
    nk = cfg.n_pcs + len(objs) + 1
    nd = np.zeros(nk, dtype=np.uint64)
    tb = np.zeros((nk, cfg.topk), dtype=np.uint64)
    tc = np.zeros((nk, cfg.topk), dtype=np.uint64)
    rc = lib().vo_approx_topk(ctypes.byref(cfg), arr, len(objs), recs.ctypes.data, len(recs), nd.ctypes.data,
                              tb.ctypes.data, tc.ctypes.data)
    if rc != 0:
        raise ValueError("vo_approx_topk rejected its arguments")
    return nd, tb, tc


def temporal_loads(cfg, objs, recs):
    """C17: uint64[n_keys, 2] = (temporal loads, temporally redundant loads) per key."""
    recs = np.ascontiguousarray(recs)
    arr, _keep = _objects(objs)
    out = np.zeros((cfg.n_pcs + len(objs) + 1, 2), dtype=np.uint64)
    if lib().vo_temporal_loads(ctypes.byref(cfg), arr, len(objs), recs.ctypes.data, len(recs), out.ctypes.data) != 0:
        raise ValueError("vo_temporal_loads rejected its arguments")
    return out


DYADIC_DTYPE = np.dtype([("state", "<u4"), ("scale", "<u4"), ("px", "<u8"), ("qx", "<u8"), ("py", "<i8"),
                         ("qy", "<i8")])


def dyadic_fit(cfg, objs, recs):
    """C21 (f2): DYADIC_DTYPE[n_keys] -- exact linear fit over the records' exact values."""
    recs = np.ascontiguousarray(recs)
    arr, _keep = _objects(objs)
    out = np.zeros(cfg.n_pcs + len(objs) + 1, dtype=DYADIC_DTYPE)
    L = lib()
    L.vo_dyadic_fit.argtypes = [ctypes.POINTER(VoConfig), ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p,
                                ctypes.c_uint64, ctypes.c_void_p]
    if L.vo_dyadic_fit(ctypes.byref(cfg), arr, len(objs), recs.ctypes.data, len(recs), out.ctypes.data) != 0:
        raise ValueError("vo_dyadic_fit rejected its arguments")
    return out


def temporal_pairs(cfg, objs, recs):
    """C17 per (PC, object): uint64[n_pcs, n_obj + 1, 2]; column n_obj = loads outside every object."""
    recs = np.ascontiguousarray(recs)
    arr, _keep = _objects(objs)
    out = np.zeros((cfg.n_pcs, len(objs) + 1, 2), dtype=np.uint64)
    L = lib()
    L.vo_temporal_pairs.argtypes = [ctypes.POINTER(VoConfig), ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p,
                                    ctypes.c_uint64, ctypes.c_void_p]
    if L.vo_temporal_pairs(ctypes.byref(cfg), arr, len(objs), recs.ctypes.data, len(recs), out.ctypes.data) != 0:
        raise ValueError("vo_temporal_pairs rejected its arguments")
    return out


def dyadic_fit_trunc(cfg, objs, recs):
    """C22 (f2): DYADIC_DTYPE[n_keys] -- C21 over the float values truncated to K mantissa bits."""
    recs = np.ascontiguousarray(recs)
    arr, _keep = _objects(objs)
    out = np.zeros(cfg.n_pcs + len(objs) + 1, dtype=DYADIC_DTYPE)
    L = lib()
    L.vo_dyadic_fit_trunc.argtypes = [ctypes.POINTER(VoConfig), ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p,
                                      ctypes.c_uint64, ctypes.c_void_p]
    if L.vo_dyadic_fit_trunc(ctypes.byref(cfg), arr, len(objs), recs.ctypes.data, len(recs), out.ctypes.data) != 0:
        raise ValueError("vo_dyadic_fit_trunc rejected its arguments")
    return out


OUTLIER_DTYPE = np.dtype([("state", "<u4"), ("scale", "<u4"), ("ax", "<u8"), ("bx", "<u8"), ("ay", "<i8"),
                          ("by", "<i8"), ("n_off", "<u8"), ("n", "<u8")])


def outlier_fit(cfg, objs, recs, flags=0):
    """C23 (f2): OUTLIER_DTYPE[n_keys] -- the interior-anchor line and the records off it."""
    recs = np.ascontiguousarray(recs)
    arr, _keep = _objects(objs)
    out = np.zeros(cfg.n_pcs + len(objs) + 1, dtype=OUTLIER_DTYPE)
    L = lib()
    L.vo_outlier_fit.argtypes = [ctypes.POINTER(VoConfig), ctypes.c_void_p, ctypes.c_uint32, ctypes.c_void_p,
                                 ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p]
    if L.vo_outlier_fit(ctypes.byref(cfg), arr, len(objs), recs.ctypes.data, len(recs), flags, out.ctypes.data) != 0:
        raise ValueError("vo_outlier_fit rejected its arguments")
    return out


# ---- C18-C20: value flow graph (layouts of ve.h's ve_api_access / ve_vfg_edge / ve_vfg_vertex)
HOST_VERTEX = 0xFFFFFFFF
ACCESS_DTYPE = np.dtype([("seq", "<u8"), ("bytes", "<u8"), ("vertex", "<u4"), ("object", "<u4"), ("mode", "<u4"),
                         ("kind", "<u4")])
VFG_EDGE_DTYPE = np.dtype([("src", "<u4"), ("dst", "<u4"), ("object", "<u4"), ("label", "<u4"), ("bytes", "<u8"),
                           ("count", "<u8")])
VFG_VERTEX_DTYPE = np.dtype([("vertex", "<u4"), ("pad", "<u4"), ("invocations", "<u8")])


def vfg_build(log):
    """C18 (Def 5.1): (edges, vertices) of an ACCESS_DTYPE log."""
    log = np.ascontiguousarray(log, dtype=ACCESS_DTYPE)
    n = len(log)
    e = np.zeros(2 * n + 1, dtype=VFG_EDGE_DTYPE)
    v = np.zeros(n + 1, dtype=VFG_VERTEX_DTYPE)
    ne, nv = ctypes.c_uint64(), ctypes.c_uint64()
    if lib().vo_vfg_build(log.ctypes.data, n, e.ctypes.data, ctypes.byref(ne), v.ctypes.data, ctypes.byref(nv)) != 0:
        raise ValueError("vo_vfg_build: an access before its allocation")
    return e[:ne.value], v[:nv.value]


def vfg_slice(edges, verts, vertex):
    """C19 (Def 5.2): the vertex slice graph of `vertex`."""
    edges, verts = np.ascontiguousarray(edges), np.ascontiguousarray(verts)
    oe = np.zeros(len(edges) + 1, dtype=VFG_EDGE_DTYPE)
    ov = np.zeros(len(verts) + 1, dtype=VFG_VERTEX_DTYPE)
    ne, nv = ctypes.c_uint64(), ctypes.c_uint64()
    lib().vo_vfg_slice(edges.ctypes.data, len(edges), verts.ctypes.data, len(verts), vertex, oe.ctypes.data,
                       ctypes.byref(ne), ov.ctypes.data, ctypes.byref(nv))
    return oe[:ne.value], ov[:nv.value]


def vfg_important(edges, verts, min_edge_bytes, min_vertex_invocations):
    """C20 (Def 5.3): the important graph."""
    edges, verts = np.ascontiguousarray(edges), np.ascontiguousarray(verts)
    oe = np.zeros(len(edges) + 1, dtype=VFG_EDGE_DTYPE)
    ov = np.zeros(len(verts) + 1, dtype=VFG_VERTEX_DTYPE)
    ne, nv = ctypes.c_uint64(), ctypes.c_uint64()
    lib().vo_vfg_important(edges.ctypes.data, len(edges), verts.ctypes.data, len(verts), min_edge_bytes,
                           min_vertex_invocations, oe.ctypes.data, ctypes.byref(ne), ov.ctypes.data, ctypes.byref(nv))
    return oe[:ne.value], ov[:nv.value]
