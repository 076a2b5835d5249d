"""CPU-side checks of the boundary: libve.so loads without a GPU and exports
every function include/ve.h declares; the generator's host and device paths
agree on layout; the product package does not reach into oracle/."""
import ctypes
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_asplos_zhouhmm022_b200")


def _declared(header):
    txt = open(header).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(ve[g]?_[a-z0-9_]+)\s*\(", txt)))


def test_libve_exports_every_declared_symbol():
    names = _declared(os.path.join(ROOT, "include", "ve.h"))
    assert "ve_analyze_records" in names and "ve_snapshot_diff" in names and "ve_object_dedup" in names
    assert "ve_merge_stats" in names and "ve_report" in names
    lib = ctypes.CDLL(os.path.join(PKG, "libve.so"))
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing
    out = subprocess.run(["nm", "-D", "--defined-only", os.path.join(PKG, "libve.so")], capture_output=True,
                         text=True).stdout
    for n in names:
        assert re.search(rf"\bT {n}\b", out), n


def test_libvegen_exports_every_declared_symbol():
    names = [n for n in _declared(os.path.join(ROOT, "include", "ve_gen.h")) if n.startswith("veg_") and
             not n.startswith(("veg_mix", "veg_h", "veg_f", "veg_t", "veg_cfg", "veg_pool", "veg_fuzz", "veg_dedup_w",
                               "veg_dedup_s", "veg_dedup_b", "veg_dedup_c"))]
    lib = ctypes.CDLL(os.path.join(ROOT, "gen", "libvegen.so"))
    missing = [n for n in names if not hasattr(lib, n)]
    assert not missing, missing


def test_product_never_touches_the_oracle():
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cc", ".cpp")):
                txt = open(os.path.join(dirpath, f)).read()
                assert not re.search(r"(import\s+oracle|from\s+oracle|#include\s*[<\"].*oracle|liboracle|ve_oracle)", txt), f
    syms = subprocess.run(["nm", "-D", os.path.join(PKG, "libve.so")], capture_output=True, text=True).stdout
    assert "vo_" not in syms and "liboracle" not in syms


def test_python_binding_fails_loudly_without_library(tmp_path, monkeypatch):
    from paper_conf_asplos_zhouhmm022_b200 import ve
    monkeypatch.setattr(ve, "_HERE", str(tmp_path))
    monkeypatch.setattr(ve, "_LIB", None)
    try:
        ve.lib()
    except RuntimeError as e:
        assert "no CPU fallback" in str(e)
    else:
        raise AssertionError("binding loaded without libve.so")


def test_record_layout():
    from paper_conf_asplos_zhouhmm022_b200 import ve
    from gen import vegen
    assert ve.RECORD_DTYPE.itemsize == 24 and vegen.REC_DTYPE == ve.RECORD_DTYPE
    assert ve.KEY_DTYPE.itemsize == 8 * (6 + 12 + 5 + 6 + 7 + 2) + 4 * 8


def test_dump_spec_layout_matches_header_struct():
    """tests/dump_spec.py packs ve_key_stats field by field in include/ve.h's order: the same values placed
    in the binding's struct mirror give the same 336 bytes (a pin of the S13 dump layout, no GPU)."""
    import numpy as np
    from paper_conf_asplos_zhouhmm022_b200 import ve
    from oracle import oracle as O
    from tests import dump_spec as D
    rng = np.random.default_rng(7)
    ok = np.zeros(1, dtype=O.KEY_DTYPE)[0]
    gk = np.zeros(1, dtype=ve.KEY_DTYPE)
    for f in ve.KEY_DTYPE.names:
        shape = ve.KEY_DTYPE[f].shape
        v = rng.integers(0, 1 << 62, size=shape if shape else None, dtype=np.int64)
        if f == "line_state":
            v = O.LINE_LINE
        if ve.KEY_DTYPE[f].base == np.dtype("<u4"):
            v = int(v) & 0xFFFFFFFF
        ok[f] = v
        gk[0][f] = v
    assert D.key_bytes(ok) == gk.tobytes() and len(gk.tobytes()) == D.KEY_BYTES
    ok["line_state"] = O.LINE_FAIL       # endpoints of a FAILed line are written as 0
    b = D.key_bytes(ok)
    assert b[30 * 8:36 * 8] == bytes(48)
