"""Field-by-field comparison of a GPU report (libve.so) with the CPU oracle.

Test infrastructure: imports nothing from the product except through the
report object handed in.  The bar is bit-exact (every field is an integer or a
bit pattern).
"""
import numpy as np

RAW_FIELDS = ["n_ld", "n_st", "n_zero", "n_ld_eq_pre", "n_st_eq_pre", "n_nosnap", "n_nan", "n_nonint",
              "n_not_f16", "n_not_bf16", "n_not_f32", "raw_min", "raw_max", "ord_min", "ord_max", "trunc_min",
              "trunc_max", "line_state", "n_distinct", "n_top"]
DERIVED = ["single_value", "single_zero", "frequent", "structured", "approx", "dict8", "heavy", "single_type"]
ENDPOINTS = ["p_x", "p_ylo", "p_yhi", "q_x", "q_ylo", "q_yhi"]
OBJ_FIELDS = ["n_elems", "n_written", "n_loaded_eq", "n_ld_reload", "n_touched"]


def compare_with_oracle(rep, okeys, oglob, oobj, max_report=50):
    """Returns a list of mismatch descriptions (empty = bit-exact parity)."""
    bad = []
    if rep.n_keys != len(okeys):
        return [f"n_keys {rep.n_keys} != {len(okeys)}"]
    g = rep.keys
    for f in RAW_FIELDS + DERIVED:
        a, b = g[f].astype(np.int64 if f == "heavy" else g[f].dtype), okeys[f].astype(g[f].dtype)
        diff = np.nonzero(g[f] != okeys[f].astype(g[f].dtype))[0]
        for k in diff[:max_report]:
            bad.append(f"key {k} {f}: gpu {g[f][k]} oracle {okeys[f][k]}")
    diff = np.nonzero((g["n_type"] != okeys["n_type"]).any(axis=1))[0]
    for k in diff[:max_report]:
        bad.append(f"key {k} n_type: gpu {list(g['n_type'][k])} oracle {list(okeys['n_type'][k])}")
    live = (okeys["line_state"] == 1) | (okeys["line_state"] == 2)
    for f in ENDPOINTS:
        diff = np.nonzero(live & (g[f] != okeys[f].astype(g[f].dtype)))[0]
        for k in diff[:max_report]:
            bad.append(f"key {k} {f}: gpu {g[f][k]} oracle {okeys[f][k]}")
    for k in range(len(okeys)):
        n = int(okeys["n_top"][k])
        gb, gc = rep.topk["bits"][k, :n], rep.topk["count"][k, :n]
        ob, oc = okeys["top_bits"][k, :n], okeys["top_count"][k, :n]
        if not (np.array_equal(gb, ob) and np.array_equal(gc, oc)):
            bad.append(f"key {k} topk: gpu {list(zip(gb, gc))} oracle {list(zip(ob, oc))}")
            if len(bad) > max_report:
                break
    for f in ("n_records", "n_invalid", "n_unmapped"):
        if int(rep.globals[f]) != int(oglob[f]):
            bad.append(f"globals {f}: gpu {rep.globals[f]} oracle {oglob[f]}")
    if len(rep.objects) != len(oobj):
        bad.append(f"n_objects {len(rep.objects)} != {len(oobj)}")
    else:
        for f in OBJ_FIELDS:
            diff = np.nonzero(rep.objects[f] != oobj[f])[0]
            for i in diff[:max_report]:
                bad.append(f"object {i} {f}: gpu {rep.objects[f][i]} oracle {oobj[f][i]}")
    return bad


def compare_diff(gd, od):
    return [f"diff {f}: gpu {gd[f]} oracle {od[f]}" for f in
            ("n_elems", "n_masked", "n_unchanged", "n_changed", "n_untouched", "redundant") if int(gd[f]) != int(od[f])]
