"""The S13 report dump as include/ve.h specifies it, built from the CPU oracle's
outputs (test infrastructure: the expected bytes of ve_report_dump come from
oracle/ only, packed in the layout the header documents).

Binary (format 0): u32 magic "VERP", version 1, n_keys, n_objects, topk;
globals (4 x u64); ve_key_stats[n_keys] (336 B); ve_topk_entry[n_keys][topk]
(entries past n_top are zero); ve_obj_stats[n_objects].  The 4th global
(hist_entries) is an implementation statistic, not a parity field: callers
mask it (GLOBALS_MASK_OFFSET).
"""
import struct

import numpy as np

from oracle import oracle as O

KEY_BYTES = 336
HEADER_BYTES = 5 * 4
GLOBALS_MASK_OFFSET = HEADER_BYTES + 3 * 8       # the hist_entries word

_SUM = ["n_ld", "n_st", "n_zero", "n_ld_eq_pre", "n_st_eq_pre", "n_nosnap"]
_FLAGS = ["n_nan", "n_nonint", "n_not_f16", "n_not_bf16", "n_not_f32"]
_MM = ["raw_min", "raw_max", "ord_min", "ord_max", "trunc_min", "trunc_max"]
_DER = ["single_value", "single_zero", "frequent", "structured", "approx", "dict8", "heavy", "single_type"]


def _live(k):
    return int(k["line_state"]) in (O.LINE_POINT, O.LINE_LINE)


def key_bytes(k):
    live = _live(k)
    ends = [int(k[f]) if live else 0 for f in ("p_x", "p_ylo", "p_yhi", "q_x", "q_ylo", "q_yhi")]
    b = struct.pack("<6Q", *[int(k[f]) for f in _SUM])
    b += struct.pack("<12Q", *[int(x) for x in k["n_type"]])
    b += struct.pack("<5Q", *[int(k[f]) for f in _FLAGS])
    b += struct.pack("<6Q", *[int(k[f]) for f in _MM])
    b += struct.pack("<Q", int(k["line_state"]))
    b += struct.pack("<QQqQQq", *ends)
    b += struct.pack("<QQ", int(k["n_distinct"]), int(k["n_top"]))
    b += struct.pack("<8I", *[int(k[f]) for f in _DER])
    assert len(b) == KEY_BYTES
    return b


def oracle_dump_bytes(okeys, oglob, oobj, topk):
    """The format-0 dump of the oracle's report (hist_entries written as 0)."""
    n_keys, n_obj = len(okeys), len(oobj)
    out = [struct.pack("<5I", 0x50524556, 1, n_keys, n_obj, topk),
           struct.pack("<4Q", int(oglob["n_records"]), int(oglob["n_invalid"]), int(oglob["n_unmapped"]), 0)]
    out += [key_bytes(k) for k in okeys]
    for k in okeys:
        n = int(k["n_top"])
        for j in range(topk):
            out.append(struct.pack("<QQ", int(k["top_bits"][j]) if j < n else 0,
                                   int(k["top_count"][j]) if j < n else 0))
    for o in oobj:
        out.append(struct.pack("<5Q", *[int(o[f]) for f in ("n_elems", "n_written", "n_loaded_eq", "n_ld_reload",
                                                                "n_touched")]))
    return b"".join(out)


def mask_hist_entries(b):
    b = bytearray(b)
    b[GLOBALS_MASK_OFFSET:GLOBALS_MASK_OFFSET + 8] = bytes(8)
    return bytes(b)


def oracle_dump_json(okeys, oglob, oobj):
    """The format-1 dump of the oracle's report, as the parsed JSON object."""
    keys = []
    for i, k in enumerate(okeys):
        live = _live(k)
        d = {"key": i}
        for f in _SUM + ["n_distinct"]:
            d[f] = int(k[f])
        for f in _DER:
            d[f] = int(k[f])
        d["heavy"] = O.TYPE_NAMES[int(k["heavy"])] if int(k["heavy"]) < 12 else "none"
        for f in _FLAGS + _MM + ["line_state"]:
            d[f] = int(k[f])
        d["p"] = [int(k["p_x"]), int(k["p_yhi"]), int(k["p_ylo"])] if live else [0, 0, 0]
        d["q"] = [int(k["q_x"]), int(k["q_yhi"]), int(k["q_ylo"])] if live else [0, 0, 0]
        d["n_type"] = [int(x) for x in k["n_type"]]
        n = int(k["n_top"])
        d["top"] = [[int(k["top_bits"][j]), int(k["top_count"][j])] for j in range(n)]
        keys.append(d)
    objs = [{"id": i, **{f: int(o[f]) for f in ("n_elems", "n_written", "n_loaded_eq", "n_ld_reload", "n_touched")}}
            for i, o in enumerate(oobj)]
    return {"n_records": int(oglob["n_records"]), "n_invalid": int(oglob["n_invalid"]),
            "n_unmapped": int(oglob["n_unmapped"]), "keys": keys, "objects": objs}


def first_difference(a, b, n_keys=None, topk=None):
    """Human-readable location of the first differing byte of two dumps."""
    if len(a) != len(b):
        return f"lengths {len(a)} != {len(b)}"
    d = np.nonzero(np.frombuffer(a, np.uint8) != np.frombuffer(b, np.uint8))[0]
    if not len(d):
        return None
    off = int(d[0])
    kb = HEADER_BYTES + 32
    if n_keys is not None and kb <= off < kb + n_keys * KEY_BYTES:
        return f"byte {off}: key {(off - kb) // KEY_BYTES} field offset {(off - kb) % KEY_BYTES}"
    return f"byte {off}"
