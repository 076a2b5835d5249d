"""Closed forms of the cfg3 (PyTorch op mix) and cfg4 (f64 stencils) workloads,
derived by hand from their construction (gen/ve_gen_core.h, SURVEY 8(d) cfg3 /
cfg4 rows).  Shared by the oracle pins (small shifts, CPU)
and the full-size GPU checks: each function takes a report-like view
(per-key arrays) and returns the list of violated closed forms.

Test infrastructure only: every expected number is arithmetic on the recipe's
sizes, or a count taken directly from the generated records.
"""
import numpy as np

from gen import vegen as G

C3_D, C3_V = 768, 30522
F64_ONE, F64_TWO = 0x3FF0000000000000, 0x4000000000000000
F32_ONE = 0x3F800000
LINE = 2


def c3_dims(shift):
    return {"T": 32768 >> shift, "M": (16 << 20) >> shift, "R": 16384 >> shift, "NI": (4 << 20) >> shift}


def c3_n(shift):
    d = c3_dims(shift)
    return (d["T"] + 2 * d["T"] * C3_D + C3_D + 3 * d["M"] + 2 * d["M"] + 3 * d["M"] + 1025 * d["R"]
            + 3 * d["NI"] + 3 * d["M"])


def c4_points(shift):
    g = 512 >> shift
    return g, g ** 3


def _chk(bad, name, got, want):
    if int(got) != int(want):
        bad.append(f"{name}: got {int(got)} want {int(want)}")


def check_cfg3(k, n_records, shift, objs):
    """k: per-key field arrays (PC keys 0..19 first, then object keys); objs: object stats."""
    d = c3_dims(shift)
    T, M, R, NI = d["T"], d["M"], d["R"], d["NI"]
    bad = []
    _chk(bad, "n_records", n_records, c3_n(shift))
    _chk(bad, "sum of PC accesses", sum(int(k["n_ld"][p]) + int(k["n_st"][p]) for p in range(20)), c3_n(shift))
    # S0 embedding: T id loads, T*D row loads, T*D stores
    _chk(bad, "PC0 n_ld", k["n_ld"][0], T)
    _chk(bad, "PC1 n_ld", k["n_ld"][1], T * C3_D)
    _chk(bad, "PC1 n_ld_eq_pre", k["n_ld_eq_pre"][1], T * C3_D)
    _chk(bad, "PC2 n_st", k["n_st"][2], T * C3_D)
    # S1 masked_fill_ of the zero padding row: 768 redundant zero stores (P14)
    _chk(bad, "PC3 n_st", k["n_st"][3], C3_D)
    _chk(bad, "PC3 n_st_eq_pre", k["n_st_eq_pre"][3], C3_D)
    _chk(bad, "PC3 single_zero", k["single_zero"][3], 1)
    # S2-S4 elementwise sizes; the `ones` operand is a single value (P9)
    for p, f in ((4, "n_ld"), (5, "n_ld"), (6, "n_st"), (7, "n_ld"), (8, "n_st"), (9, "n_ld"), (10, "n_ld"),
                 (11, "n_st")):
        _chk(bad, f"PC{p} {f}", k[f][p], M)
    _chk(bad, "PC10 single_value", k["single_value"][10], 1)
    _chk(bad, "PC10 n_ld_eq_pre", k["n_ld_eq_pre"][10], M)
    _chk(bad, "PC10 top value", k["top_bits"][10][0], F32_ONE)
    _chk(bad, "PC10 top count", k["top_count"][10][0], M)
    # S5 reduce: 1024 loads per row and one store per row
    _chk(bad, "PC12 n_ld", k["n_ld"][12], 1024 * R)
    _chk(bad, "PC12 n_ld_eq_pre", k["n_ld_eq_pre"][12], 1024 * R)
    _chk(bad, "PC13 n_st", k["n_st"][13], R)
    # S6 index_select: the i64 arange index is an exact line through (idx_base + 8 i, i)
    o11 = G.objects(G.scaled(G.CFG3, shift))[11]
    _chk(bad, "PC14 n_ld", k["n_ld"][14], NI)
    _chk(bad, "PC14 line_state", k["line_state"][14], LINE)
    _chk(bad, "PC14 p_x", k["p_x"][14], o11["base"])
    _chk(bad, "PC14 p_y", k["p_ylo"][14], 0)
    _chk(bad, "PC14 q_x", k["q_x"][14], o11["base"] + 8 * (NI - 1))
    _chk(bad, "PC14 q_y", k["q_ylo"][14], NI - 1)
    # S7 zeros_like + zero_ over a zero grad, ones fill over ones: all redundant (P10)
    for p in (17, 18, 19):
        _chk(bad, f"PC{p} n_st", k["n_st"][p], M)
        _chk(bad, f"PC{p} n_st_eq_pre", k["n_st_eq_pre"][p], M)
    _chk(bad, "PC17 single_zero", k["single_zero"][17], 1)
    _chk(bad, "PC19 single_value", k["single_value"][19], 1)
    # object keys (n_pcs + id): emb weight loaded T*D times, written 768 times
    _chk(bad, "obj emb_w n_ld", k["n_ld"][20 + 0], T * C3_D)
    _chk(bad, "obj emb_w n_st", k["n_st"][20 + 0], C3_D)
    _chk(bad, "obj grad n_st_eq_pre", k["n_st_eq_pre"][20 + 14], 2 * M)
    # elementwise operands: every element read once, nothing reloaded
    for i in (3, 4, 7, 9, 11, 12):
        _chk(bad, f"obj {i} n_ld_reload", objs["n_ld_reload"][i], 0)
    return bad


def check_cfg4(k, n_records, shift, epoch, objs):
    g, P = c4_points(shift)
    bad = []
    tw = (P + 19) // 20                       # points with a != 1 (p % 20 == 0)
    if epoch == 0:
        _chk(bad, "n_records", n_records, 8 * P)
        for p in range(7):
            _chk(bad, f"PC{p} n_ld", k["n_ld"][p], P)
            _chk(bad, f"PC{p} n_ld_eq_pre", k["n_ld_eq_pre"][p], P)
            _chk(bad, f"PC{p} approx", k["approx"][p], 1)     # one K=7 bucket [300, 302) (P7)
        _chk(bad, "PC7 n_st", k["n_st"][7], P)
        _chk(bad, "PC7 n_st_eq_pre", k["n_st_eq_pre"][7], 0)
        _chk(bad, "PC7 approx", k["approx"][7], 1)
        _chk(bad, "T_in n_ld_reload", objs["n_ld_reload"][0], 6 * P)   # 7 loads per element, 1 first read
        _chk(bad, "T_out n_written", objs["n_written"][1], P)
        if int(k["n_distinct"][0]) > 4096:
            bad.append(f"PC0 n_distinct {int(k['n_distinct'][0])} > 4096")
    else:
        _chk(bad, "n_records", n_records, 7 * P)
        o = G.objects(G.scaled(G.CFG4, shift), 1)
        for p in range(8, 14):
            _chk(bad, f"PC{p} n_ld", k["n_ld"][p], P)
        # a: 1.0 except every 20th point (P11); frequent value 1.0
        _chk(bad, "PC8 n_distinct", k["n_distinct"][8], 2)
        _chk(bad, "PC8 top0", k["top_bits"][8][0], F64_ONE)
        _chk(bad, "PC8 top0 count", k["top_count"][8][0], P - tw)
        _chk(bad, "PC8 top1", k["top_bits"][8][1], F64_TWO)
        _chk(bad, "PC8 top1 count", k["top_count"][8][1], tw)
        _chk(bad, "PC8 frequent", k["frequent"][8], 1)
        # xc[x] = x + 64: an exact line through the xc array
        _chk(bad, "PC9 line_state", k["line_state"][9], LINE)
        _chk(bad, "PC9 p_x", k["p_x"][9], o[5]["base"])
        _chk(bad, "PC9 p_y", k["p_ylo"][9], 64)
        _chk(bad, "PC9 q_x", k["q_x"][9], o[5]["base"] + 8 * (g - 1))
        _chk(bad, "PC9 q_y", k["q_ylo"][9], g - 1 + 64)
        _chk(bad, "PC9 n_distinct", k["n_distinct"][9], g)
        # vol == 1.0 everywhere: single value
        _chk(bad, "PC10 single_value", k["single_value"][10], 1)
        # s stores equal the pre value wherever a == 1 (redundant stores)
        _chk(bad, "PC14 n_st", k["n_st"][14], P)
        _chk(bad, "PC14 n_st_eq_pre", k["n_st_eq_pre"][14], P - tw)
        _chk(bad, "s n_ld_reload", objs["n_ld_reload"][3], 2 * P)       # 3 loads per element
        _chk(bad, "xc n_ld_reload", objs["n_ld_reload"][5], P - g)
        _chk(bad, "a n_ld_reload", objs["n_ld_reload"][2], 0)
    return bad
