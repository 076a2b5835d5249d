"""Thin ctypes binding of libve.so (include/ve.h): argument marshalling only.

Every step of the analysis runs in libve.so's CUDA kernels; there is no CPU
fallback -- importing this module on a box without the built library, or
calling it without a CUDA device, fails loudly.  torch is used only for device
memory and streams.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

OK, ERR_INVALID, ERR_CUDA, ERR_NOMEM, ERR_CAPACITY, ERR_NCCL, ERR_STATE = range(7)
DIFF_WRITTEN, DIFF_ALL, DIFF_MASK = 0, 1, 2
LINE_EMPTY, LINE_POINT, LINE_LINE, LINE_FAIL = 0, 1, 2, 3
STATUS_NAMES = ["VE_OK", "VE_ERR_INVALID", "VE_ERR_CUDA", "VE_ERR_NOMEM", "VE_ERR_CAPACITY", "VE_ERR_NCCL",
                "VE_ERR_STATE"]

RECORD_DTYPE = np.dtype([("addr", "<u8"), ("value", "<u8"), ("pc", "<u4"), ("meta", "<u4")])

# mirror of ve_key_stats
KEY_DTYPE = np.dtype(
    [(f, "<u8") for f in ("n_ld", "n_st", "n_zero", "n_ld_eq_pre", "n_st_eq_pre", "n_nosnap")]
    + [("n_type", "<u8", (12,))]
    + [(f, "<u8") for f in ("n_nan", "n_nonint", "n_not_f16", "n_not_bf16", "n_not_f32")]
    + [(f, "<u8") for f in ("raw_min", "raw_max", "ord_min", "ord_max", "trunc_min", "trunc_max")]
    + [("line_state", "<u8"), ("p_x", "<u8"), ("p_ylo", "<u8"), ("p_yhi", "<i8"), ("q_x", "<u8"),
       ("q_ylo", "<u8"), ("q_yhi", "<i8"), ("n_distinct", "<u8"), ("n_top", "<u8")]
    + [(f, "<u4") for f in ("single_value", "single_zero", "frequent", "structured", "approx", "dict8", "heavy",
                            "single_type")])
TOPK_DTYPE = np.dtype([("bits", "<u8"), ("count", "<u8")])
OBJ_DTYPE = np.dtype([(f, "<u8") for f in ("n_elems", "n_written", "n_loaded_eq", "n_ld_reload", "n_touched")])
GLOB_DTYPE = np.dtype([(f, "<u8") for f in ("n_records", "n_invalid", "n_unmapped", "hist_entries")])
INTERVAL_DTYPE = np.dtype([("start", "<u8"), ("end", "<u8")])   # ve_interval (inclusive)
COPY_NONE, COPY_SEGMENT, COPY_MINMAX = 0, 1, 2
# value flow graph (ve_api_access / ve_vfg_edge / ve_vfg_vertex)
HOST_VERTEX = 0xFFFFFFFF
ACC_READ, ACC_WRITE = 1, 2
EV_DEVICE, EV_ALLOC, EV_H2D, EV_D2H = 0, 1, 2, 3
ACCESS_DTYPE = np.dtype([("seq", "<u8"), ("bytes", "<u8"), ("vertex", "<u4"), ("object", "<u4"), ("mode", "<u4"),
                         ("kind", "<u4")])
VFG_EDGE_DTYPE = np.dtype([("src", "<u4"), ("dst", "<u4"), ("object", "<u4"), ("label", "<u4"), ("bytes", "<u8"),
                           ("count", "<u8")])
VFG_VERTEX_DTYPE = np.dtype([("vertex", "<u4"), ("pad", "<u4"), ("invocations", "<u8")])
PLAN_DTYPE = np.dtype([(f, "<u8") for f in ("n_segments", "accessed_bytes", "lo", "hi", "direct_bytes",
                                           "minmax_bytes")] + [("choice", "<u4"), ("pad", "<u4")])
DIFF_DTYPE = np.dtype([(f, "<u8") for f in ("n_elems", "n_masked", "n_unchanged", "n_changed", "n_untouched")]
                      + [("redundant", "<u4"), ("pad", "<u4")])


DYADIC_DTYPE = np.dtype([("state", "<u4"), ("scale", "<u4"), ("px", "<u8"), ("qx", "<u8"), ("py", "<i8"),
                         ("qy", "<i8")])
OUTLIER_DTYPE = np.dtype([("state", "<u4"), ("scale", "<u4"), ("ax", "<u8"), ("bx", "<u8"), ("ay", "<i8"),
                          ("by", "<i8"), ("n_off", "<u8"), ("n", "<u8")])
FIT_TRUNC = 1


class VeError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES[status] if 0 <= status < 7 else status}: {msg}")
        self.status = status


class _Config(ctypes.Structure):
    _fields_ = [("n_pcs", ctypes.c_uint32), ("max_objects", ctypes.c_uint32), ("topk", ctypes.c_uint32),
                ("mant_bits", ctypes.c_uint32), ("t_redundant_pct", ctypes.c_uint32),
                ("t_frequent_pct", ctypes.c_uint32), ("hist_capacity", ctypes.c_uint64),
                ("min_windows_per_warp", ctypes.c_uint32), ("reserved", ctypes.c_uint32)]


class _Unit(ctypes.Structure):
    _fields_ = [("d_records", ctypes.c_void_p), ("n", ctypes.c_uint64), ("pc_base", ctypes.c_uint32),
                ("n_pcs", ctypes.c_uint32)]


class _Object(ctypes.Structure):
    _fields_ = [("base", ctypes.c_uint64), ("size", ctypes.c_uint64), ("pre", ctypes.c_void_p),
                ("post", ctypes.c_void_p), ("id", ctypes.c_uint32), ("elem_width", ctypes.c_uint32)]


def lib():
    global _LIB
    if _LIB is None:
        path = os.environ.get("VE_LIB_PATH") or os.path.join(_HERE, "libve.so")   # override: A/B of builds
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run __graft_entry__.build() (no CPU fallback exists)")
        L = ctypes.CDLL(path)
        vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        st = ctypes.c_int
        sig = {
            "ve_create": ([ctypes.POINTER(_Config), i32, ctypes.POINTER(vp)], st),
            "ve_destroy": ([vp], st),
            "ve_last_error": ([vp], ctypes.c_char_p),
            "ve_set_objects": ([vp, vp, u32], st),
            "ve_reset": ([vp], st),
            "ve_analyze_records": ([vp, vp, u64, vp], st),
            "ve_analyze_records_host": ([vp, vp, u64, vp], st),
            "ve_snapshot_diff": ([vp, u32, u32, vp, vp, vp], st),
            "ve_object_dedup": ([vp, vp, u32, vp, vp], st),
            "ve_merge_stats": ([vp, vp, vp, vp], st),
            "ve_report": ([vp, ctypes.POINTER(vp)], st),
            "ve_report_free": ([vp], None),
            "ve_report_n_keys": ([vp], u32),
            "ve_report_n_objects": ([vp], u32),
            "ve_report_topk": ([vp], u32),
            "ve_report_keys": ([vp, vp], st),
            "ve_report_topk_entries": ([vp, vp], st),
            "ve_report_objects": ([vp, vp], st),
            "ve_report_globals": ([vp, vp], st),
            "ve_report_dump": ([vp, ctypes.c_char_p, i32], st),
            "ve_kernel_launches": ([], u64),
            "ve_merge_group": ([ctypes.POINTER(vp), u32, vp], st),
            "ve_nccl_get_unique_id": ([vp], st),
            "ve_nccl_comm_init": ([ctypes.POINTER(vp), i32, vp, i32], st),
            "ve_nccl_comm_destroy": ([vp], st),
            "ve_interval_merge": ([vp, vp, u64, vp, ctypes.POINTER(u64), vp], st),
            "ve_approx_topk": ([vp, vp, vp, vp], st),
            "ve_temporal_loads": ([vp, vp, u64, vp, vp], st),
            "ve_dyadic_fit": ([vp, vp, u64, vp, vp], st),
            "ve_vfg_build": ([vp, u64, ctypes.POINTER(vp)], st),
            "ve_vfg_slice": ([vp, u32, ctypes.POINTER(vp)], st),
            "ve_vfg_important": ([vp, u64, u64, ctypes.POINTER(vp)], st),
            "ve_vfg_size": ([vp, ctypes.POINTER(u64), ctypes.POINTER(u64)], st),
            "ve_vfg_vertices": ([vp, vp], st),
            "ve_vfg_edges": ([vp, vp], st),
            "ve_vfg_free": ([vp], None),
            "ve_record_intervals": ([vp, vp, u64, vp, ctypes.POINTER(u64), vp], st),
            "ve_plan_copies": ([vp, vp, u64, u32, u32, vp, vp], st),
            "ve_snapshot_diff_all": ([vp, u32, vp, vp, vp], st),
            "ve_dyadic_fit_ex": ([vp, vp, u64, u32, vp, vp], st),
            "ve_temporal_loads_ex": ([vp, vp, u64, vp, vp, vp], st),
            "ve_outlier_fit": ([vp, vp, u64, u32, vp, vp], st),
            "ve_object_dedup_comm": ([vp, vp, u32, vp, vp, vp], st),
            "ve_snapshot_diff_all_group": ([ctypes.POINTER(vp), u32, u32, vp, vp], st),
            "ve_object_dedup_group": ([ctypes.POINTER(vp), u32, vp, u32, vp, vp], st),
            "ve_set_units": ([vp, vp, u32, vp, u32], st),
            "ve_analyze_units": ([vp, vp, u32, vp], st),
        }
        for name, (args, res) in sig.items():
            if os.environ.get("VE_LIB_PATH") and not hasattr(L, name):
                continue          # (an older build under A/B timing: calls it lacks are not made)
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _LIB = L
    return _LIB


def _ptr(x):
    """device/host pointer of a torch tensor, numpy array or int"""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if isinstance(x, np.ndarray):
        return x.ctypes.data
    raise TypeError(type(x))


def _stream(stream):
    if stream is None:
        try:
            import torch
            if torch.cuda.is_available():
                return torch.cuda.current_stream().cuda_stream
        except ImportError:
            pass
        return 0
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def kernel_launches():
    """libve kernels launched by this process so far (ve_kernel_launches)."""
    return lib().ve_kernel_launches()


def rank_chunk(n, rank, world):
    """[lo, hi) of the contiguous share of n records analyzed by `rank` of `world` (strong scaling)."""
    return n * rank // world, n * (rank + 1) // world


def lpt_assign(costs, world):
    """Rank of each unit under longest-processing-time-first (cfg5's independent
    kernels by record count): units in decreasing cost (ties by index) go to the least-loaded rank
    (ties by rank).  Deterministic, so every rank computes the same plan without communication;
    max load <= (4/3 - 1/(3 world)) x the optimum (Graham's bound)."""
    import heapq
    order = sorted(range(len(costs)), key=lambda i: (-int(costs[i]), i))
    heap = [(0, r) for r in range(world)]
    owner = [0] * len(costs)
    for i in order:
        load, r = heapq.heappop(heap)
        owner[i] = r
        heapq.heappush(heap, (load + int(costs[i]), r))
    return owner


class ValueFlowGraph:
    """ve_vfg_* (Defs 5.1-5.3): built from an ACCESS_DTYPE log in program order (host-side, no device)."""

    def __init__(self, handle):
        self._h = handle
        nv, ne = ctypes.c_uint64(), ctypes.c_uint64()
        lib().ve_vfg_size(handle, ctypes.byref(nv), ctypes.byref(ne))
        self.vertices = np.zeros(nv.value, dtype=VFG_VERTEX_DTYPE)
        self.edges = np.zeros(ne.value, dtype=VFG_EDGE_DTYPE)
        lib().ve_vfg_vertices(handle, self.vertices.ctypes.data if nv.value else None)
        lib().ve_vfg_edges(handle, self.edges.ctypes.data if ne.value else None)

    @classmethod
    def build(cls, log):
        log = np.ascontiguousarray(log, dtype=ACCESS_DTYPE)
        h = ctypes.c_void_p()
        rc = lib().ve_vfg_build(log.ctypes.data if len(log) else None, len(log), ctypes.byref(h))
        if rc != OK:
            raise VeError(rc, "ve_vfg_build: seq not in program order or an access before its allocation")
        return cls(h)

    def slice(self, vertex):
        h = ctypes.c_void_p()
        rc = lib().ve_vfg_slice(self._h, vertex, ctypes.byref(h))
        if rc != OK:
            raise VeError(rc, f"ve_vfg_slice: no vertex {vertex}")
        return ValueFlowGraph(h)

    def important(self, min_edge_bytes, min_vertex_invocations):
        h = ctypes.c_void_p()
        rc = lib().ve_vfg_important(self._h, min_edge_bytes, min_vertex_invocations, ctypes.byref(h))
        if rc != OK:
            raise VeError(rc, "ve_vfg_important")
        return ValueFlowGraph(h)

    def __del__(self):
        if getattr(self, "_h", None) and _LIB is not None:
            _LIB.ve_vfg_free(self._h)
            self._h = None


def merge_group(contexts, stream=None):
    """ve_merge_group: merge same-device contexts with the rank-merge algorithm (context i = rank i)."""
    arr = (ctypes.c_void_p * len(contexts))(*[c.handle.value for c in contexts])
    rc = lib().ve_merge_group(arr, len(contexts), _stream(stream))
    if rc != OK:
        raise VeError(rc, "ve_merge_group: " + lib().ve_last_error(contexts[0].handle).decode())


def _objects_arr(objs):
    arr = (_Object * max(len(objs), 1))()
    for i, o in enumerate(objs):
        arr[i] = _Object(o["base"], o["size"], _ptr(o.get("pre")), _ptr(o.get("post")), o["id"], o.get("elem_width", 8))
    return arr


def snapshot_diff_all_group(contexts, mode=DIFF_WRITTEN, stream=None):
    """ve_snapshot_diff_all_group: the object-sharded diff with context i playing rank i (one device)."""
    arr = (ctypes.c_void_p * len(contexts))(*[c.handle.value for c in contexts])
    n = getattr(contexts[0], "n_objects", 0)
    out = np.zeros(max(n, 1), dtype=DIFF_DTYPE)
    rc = lib().ve_snapshot_diff_all_group(arr, len(contexts), mode, out.ctypes.data, _stream(stream))
    if rc != OK:
        raise VeError(rc, "ve_snapshot_diff_all_group: " + lib().ve_last_error(contexts[0].handle).decode())
    return out[:n]


def object_dedup_group(contexts, objs, stream=None):
    """ve_object_dedup_group: the object-sharded duplicate scan with context i playing rank i."""
    arr = (ctypes.c_void_p * len(contexts))(*[c.handle.value for c in contexts])
    g = np.zeros(max(len(objs), 1), dtype=np.uint32)
    rc = lib().ve_object_dedup_group(arr, len(contexts), _objects_arr(objs), len(objs), g.ctypes.data, _stream(stream))
    if rc != OK:
        raise VeError(rc, "ve_object_dedup_group: " + lib().ve_last_error(contexts[0].handle).decode())
    return g[:len(objs)]


def nccl_unique_id():
    buf = (ctypes.c_uint8 * 128)()
    rc = lib().ve_nccl_get_unique_id(buf)
    if rc != OK:
        raise VeError(rc, "ve_nccl_get_unique_id")
    return bytes(buf)


def nccl_comm_init(uid, rank, world):
    comm = ctypes.c_void_p()
    buf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
    rc = lib().ve_nccl_comm_init(ctypes.byref(comm), world, buf, rank)
    if rc != OK:
        raise VeError(rc, "ve_nccl_comm_init")
    return comm.value


def nccl_comm_from_torch(rank, world, group=None):
    """One NCCL communicator over the torch.distributed ranks: rank 0 creates the unique id,
    torch.distributed broadcasts it (any backend), every rank joins."""
    import torch
    import torch.distributed as dist
    uid = torch.zeros(128, dtype=torch.uint8)
    if rank == 0:
        uid = torch.tensor(list(nccl_unique_id()), dtype=torch.uint8)
    if dist.get_backend(group) == "nccl":
        uid = uid.cuda()
    dist.broadcast(uid, src=0, group=group)
    return nccl_comm_init(bytes(uid.cpu().tolist()), rank, world)


class Report:
    """Host copy of a ve_report: keys (KEY_DTYPE), topk[n_keys, k] (TOPK_DTYPE), objects, globals."""

    def __init__(self, handle):
        L = lib()
        self.n_keys = L.ve_report_n_keys(handle)
        self.n_objects = L.ve_report_n_objects(handle)
        self.k = L.ve_report_topk(handle)
        self.keys = np.zeros(self.n_keys, dtype=KEY_DTYPE)
        self.topk = np.zeros((self.n_keys, self.k), dtype=TOPK_DTYPE)
        self.objects = np.zeros(max(self.n_objects, 1), dtype=OBJ_DTYPE)
        g = np.zeros(1, dtype=GLOB_DTYPE)
        L.ve_report_keys(handle, self.keys.ctypes.data)
        L.ve_report_topk_entries(handle, self.topk.ctypes.data)
        L.ve_report_objects(handle, self.objects.ctypes.data)
        L.ve_report_globals(handle, g.ctypes.data)
        self.objects = self.objects[:self.n_objects]
        self.globals = g[0]
        self._handle = handle

    def dump(self, path, fmt=1):
        rc = lib().ve_report_dump(self._handle, path.encode(), fmt)
        if rc != OK:
            raise VeError(rc, "ve_report_dump")

    def close(self):
        if self._handle:
            lib().ve_report_free(self._handle)
            self._handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Context:
    """A ve_ctx bound to one CUDA device."""

    def __init__(self, n_pcs, max_objects=64, topk=8, mant_bits=7, t_redundant_pct=33, t_frequent_pct=33,
                 hist_capacity=1 << 22, device=None, min_windows_per_warp=0):
        L = lib()
        if device is None:
            import torch
            device = torch.cuda.current_device()
        self.device = device
        cfg = _Config(n_pcs, max_objects, topk, mant_bits, t_redundant_pct, t_frequent_pct, hist_capacity,
                      min_windows_per_warp, 0)
        h = ctypes.c_void_p()
        rc = L.ve_create(ctypes.byref(cfg), device, ctypes.byref(h))
        if rc != OK:
            raise VeError(rc, "ve_create")
        self._h = h
        self.n_pcs = n_pcs
        self.topk = topk
        self._keep = []

    def _check(self, rc, what):
        if rc != OK:
            raise VeError(rc, f"{what}: {lib().ve_last_error(self._h).decode()}")

    @property
    def handle(self):
        return self._h

    def set_objects(self, objs):
        """objs: dicts {base, size, id, elem_width, pre, post} (pre/post: device tensors/pointers or None)."""
        arr = (_Object * max(len(objs), 1))()
        keep = []
        for i, o in enumerate(objs):
            arr[i] = _Object(o["base"], o["size"], _ptr(o.get("pre")), _ptr(o.get("post")), o["id"],
                             o["elem_width"])
            keep += [o.get("pre"), o.get("post")]
        self._keep = keep
        self._check(lib().ve_set_objects(self._h, arr, len(objs)), "ve_set_objects")
        self.n_objects = len(objs)

    def set_units(self, units_objs):
        """units_objs: one list of object dicts per unit (ids unique over the whole set)."""
        flat = [o for objs in units_objs for o in objs]
        arr = (_Object * max(len(flat), 1))()
        keep = []
        for i, o in enumerate(flat):
            arr[i] = _Object(o["base"], o["size"], _ptr(o.get("pre")), _ptr(o.get("post")), o["id"],
                             o["elem_width"])
            keep += [o.get("pre"), o.get("post")]
        cnt = (ctypes.c_uint32 * max(len(units_objs), 1))(*[len(objs) for objs in units_objs])
        self._keep = keep
        self._check(lib().ve_set_units(self._h, arr, len(flat), cnt, len(units_objs)), "ve_set_units")
        self.n_objects = len(flat)

    def analyze_units(self, units, stream=None):
        """units: (d_records, n, pc_base, n_pcs) per unit, in ve_set_units' order."""
        arr = (_Unit * max(len(units), 1))()
        for i, (d, n, pcb, npc) in enumerate(units):
            arr[i] = _Unit(_ptr(d), n, pcb, npc)
        self._check(lib().ve_analyze_units(self._h, arr, len(units), _stream(stream)), "ve_analyze_units")

    def reset(self):
        self._check(lib().ve_reset(self._h), "ve_reset")

    def analyze_records(self, d_records, n=None, stream=None):
        if n is None:
            n = d_records.numel() // 24 if hasattr(d_records, "numel") else len(d_records)
        self._check(lib().ve_analyze_records(self._h, _ptr(d_records), n, _stream(stream)), "ve_analyze_records")

    def analyze_records_host(self, h_records, n=None, stream=None):
        if n is None:
            n = len(h_records) if isinstance(h_records, np.ndarray) and h_records.dtype.itemsize == 24 else \
                h_records.numel() // 24
        self._check(lib().ve_analyze_records_host(self._h, _ptr(h_records), n, _stream(stream)),
                    "ve_analyze_records_host")

    def snapshot_diff(self, obj_id, mode=DIFF_WRITTEN, d_mask=None, stream=None):
        out = np.zeros(1, dtype=DIFF_DTYPE)
        self._check(lib().ve_snapshot_diff(self._h, obj_id, mode, _ptr(d_mask), out.ctypes.data, _stream(stream)),
                    "ve_snapshot_diff")
        return out[0]

    def object_dedup(self, objs, comm=None, stream=None):
        """ve_object_dedup (comm: ve_object_dedup_comm, sharded over the ranks of an NCCL comm)."""
        arr = _objects_arr(objs)
        g = np.zeros(max(len(objs), 1), dtype=np.uint32)
        if comm:
            self._check(lib().ve_object_dedup_comm(self._h, arr, len(objs), ctypes.c_void_p(comm), g.ctypes.data,
                                                   _stream(stream)), "ve_object_dedup_comm")
        else:
            self._check(lib().ve_object_dedup(self._h, arr, len(objs), g.ctypes.data, _stream(stream)),
                        "ve_object_dedup")
        return g[:len(objs)]

    def snapshot_diff_all(self, mode=DIFF_WRITTEN, comm=None, stream=None):
        """ve_snapshot_diff_all: DIFF_DTYPE[n_objects] (by id) of every object with both snapshots,
        sharded by object over the ranks of an NCCL comm (None: this rank alone)."""
        n = getattr(self, "n_objects", 0)
        out = np.zeros(max(n, 1), dtype=DIFF_DTYPE)
        self._check(lib().ve_snapshot_diff_all(self._h, mode, ctypes.c_void_p(comm) if comm else None,
                                               out.ctypes.data, _stream(stream)), "ve_snapshot_diff_all")
        return out[:n]

    def merge(self, other=None, comm=None, stream=None):
        """ve_merge_stats: with another same-device context, or over all ranks of an NCCL comm."""
        self._check(lib().ve_merge_stats(self._h, other._h if other is not None else None,
                                         ctypes.c_void_p(comm) if comm else None, _stream(stream)),
                    "ve_merge_stats")

    def approx_topk(self, stream=None):
        """ve_approx_topk: (ndistinct[n_keys], top[n_keys, topk] of TOPK_DTYPE) of the truncated values."""
        nk = self.n_pcs + getattr(self, "n_objects", 0) + 1
        nd = np.zeros(nk, dtype=np.uint64)
        top = np.zeros(nk * self.topk, dtype=TOPK_DTYPE)
        self._check(lib().ve_approx_topk(self._h, nd.ctypes.data, top.ctypes.data, _stream(stream)),
                    "ve_approx_topk")
        return nd, top.reshape(nk, self.topk)

    def dyadic_fit(self, d_records, n, stream=None):
        """ve_dyadic_fit: DYADIC_DTYPE[n_keys] -- exact linear fit over the records' exact values (f2)."""
        nk = self.n_pcs + getattr(self, "n_objects", 0) + 1
        out = np.zeros(nk, dtype=DYADIC_DTYPE)
        self._check(lib().ve_dyadic_fit(self._h, _ptr(d_records), n, out.ctypes.data, _stream(stream)),
                    "ve_dyadic_fit")
        return out

    def dyadic_fit_trunc(self, d_records, n, stream=None):
        """ve_dyadic_fit_ex(VE_FIT_TRUNC): C22, the fit over the K-bit truncated float values (f2)."""
        nk = self.n_pcs + getattr(self, "n_objects", 0) + 1
        out = np.zeros(nk, dtype=DYADIC_DTYPE)
        self._check(lib().ve_dyadic_fit_ex(self._h, _ptr(d_records), n, FIT_TRUNC, out.ctypes.data, _stream(stream)),
                    "ve_dyadic_fit_ex")
        return out

    def outlier_fit(self, d_records, n, flags=0, stream=None):
        """ve_outlier_fit: C23, OUTLIER_DTYPE[n_keys] -- interior-anchor line and records off it (f2)."""
        nk = self.n_pcs + getattr(self, "n_objects", 0) + 1
        out = np.zeros(nk, dtype=OUTLIER_DTYPE)
        self._check(lib().ve_outlier_fit(self._h, _ptr(d_records), n, flags, out.ctypes.data, _stream(stream)),
                    "ve_outlier_fit")
        return out

    def temporal_loads(self, d_records, n, stream=None):
        """ve_temporal_loads: uint64[n_keys, 2] = (temporal, temporally redundant) loads per key."""
        nk = self.n_pcs + getattr(self, "n_objects", 0) + 1
        out = np.zeros((nk, 2), dtype=np.uint64)
        self._check(lib().ve_temporal_loads(self._h, _ptr(d_records), n, out.ctypes.data, _stream(stream)),
                    "ve_temporal_loads")
        return out

    def temporal_pairs(self, d_records, n, stream=None):
        """ve_temporal_loads_ex: (uint64[n_keys, 2] per key, uint64[n_pcs, n_objects + 1, 2] per (PC, object))."""
        nk = self.n_pcs + getattr(self, "n_objects", 0) + 1
        out = np.zeros((nk, 2), dtype=np.uint64)
        pairs = np.zeros((self.n_pcs, getattr(self, "n_objects", 0) + 1, 2), dtype=np.uint64)
        self._check(lib().ve_temporal_loads_ex(self._h, _ptr(d_records), n, out.ctypes.data, pairs.ctypes.data,
                                               _stream(stream)), "ve_temporal_loads_ex")
        return out, pairs

    def interval_merge(self, d_in, n, d_out, stream=None):
        """ve_interval_merge: merge n device intervals (16 B each) into d_out; returns the merged count."""
        m = ctypes.c_uint64(0)
        self._check(lib().ve_interval_merge(self._h, _ptr(d_in), n, _ptr(d_out), ctypes.byref(m), _stream(stream)),
                    "ve_interval_merge")
        return m.value

    def record_intervals(self, d_records, n, d_out, stream=None):
        """ve_record_intervals: merged byte intervals accessed by n device records; returns the count."""
        m = ctypes.c_uint64(0)
        self._check(lib().ve_record_intervals(self._h, _ptr(d_records), n, _ptr(d_out), ctypes.byref(m),
                                              _stream(stream)), "ve_record_intervals")
        return m.value

    def plan_copies(self, d_merged, n, seg_max=32, dense_pct=50, stream=None):
        """ve_plan_copies: per-object adaptive copy plan (PLAN_DTYPE, indexed by object id)."""
        out = np.zeros(max(getattr(self, "n_objects", 0), 1), dtype=PLAN_DTYPE)
        self._check(lib().ve_plan_copies(self._h, _ptr(d_merged), n, seg_max, dense_pct, out.ctypes.data,
                                         _stream(stream)), "ve_plan_copies")
        return out[:getattr(self, "n_objects", 0)]

    def report(self):
        h = ctypes.c_void_p()
        self._check(lib().ve_report(self._h, ctypes.byref(h)), "ve_report")
        return Report(h)

    def close(self):
        if getattr(self, "_h", None):
            lib().ve_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
