"""Closed forms of the cfg5 kernel set (SURVEY 8(d) cfg5 "Kernels"; generator:
gen/ve_gen_core.h veg_cfg5_record / veg_c5_elem), derived from the recipe, not
from either implementation: per PC, the record counts, the load/store split and
the pre-snapshot matches that follow from cfg1's 16 PC roles, and the values of
the constant roles.  Used to pin the oracle on scaled kernels
(tests/test_oracle_cfg5.py) and to check full-size GPU reports where running the
oracle is not allowed (bench.py) or too slow (every kernel of the 10^9 records).

cfg1 roles (gen/ve_gen_core.h veg_cfg1_value / veg_cfg1_pre): 0..7 are loads whose
pre value equals the loaded value; 8..15 are stores; pre of a store element is
0 for roles 8, 11, 13, the value itself on even elements (value ^ 1 on odd ones)
for role 9, and value ^ 1 otherwise.  Role 0 loads 0, role 1 loads 0x2A, role 8
stores 0; role 11 stores 0 except on elements e % 250 == 0 (a non-zero f32);
role 13 stores +0.0 on even and -0.0 on odd elements.
"""
import numpy as np

from gen import vegen as G


def geometry(cfg, k):
    inf = G.info(cfg, k)
    n, P, O = inf["n_records"], inf["n_pcs"], inf["n_obj"]
    L = 32 * (((n + 31) // 32 + P - 1) // P)
    return n, P, O, L


def pc_elements(n, P, O, L, p):
    """element indices (in object p % O) of the records of PC p, in record order"""
    r = np.arange(n, dtype=np.int64)
    g = r // 32
    r = r[g % P == p]
    g = r // 32
    return (p // O) * L + (g // P) * 32 + r % 32


def expected(cfg, k, roles):
    """{pc: dict of closed-form fields}; roles[p] = cfg1 role of PC p (veg_c5_role)."""
    n, P, O, L = geometry(cfg, k)
    out = {}
    for p in range(P):
        e = pc_elements(n, P, O, L, p)
        role, c = roles[p], len(e)
        d = {"n_ld": c if role < 8 else 0, "n_st": c if role >= 8 else 0,
             "n_ld_eq_pre": c if role < 8 else 0}
        if role in (8,):
            d["n_st_eq_pre"] = c
        elif role == 11:
            d["n_st_eq_pre"] = int(np.count_nonzero(e % 250 != 0))
        elif role in (9, 13):
            d["n_st_eq_pre"] = int(np.count_nonzero(e % 2 == 0))
        else:
            d["n_st_eq_pre"] = 0
        if role in (0, 8) and c:
            d["raw_min"] = d["raw_max"] = 0
            d["single_zero"] = 1
        if role == 1 and c:
            d["raw_min"] = d["raw_max"] = 0x2A
            d["single_value"] = 1
        out[p] = d
    return out


def roles_of(k, P):
    """veg_c5_role restated from the recipe: splitmix64-based draw from the fixed geometry seed 5"""
    return [int(G.c5_role(k, p)) for p in range(P)]


def check_cfg5_kernel(keys, n_records, cfg, k):
    """keys: per-key arrays (oracle or GPU report, PC keys first); returns mismatch strings."""
    n, P, O, L = geometry(cfg, k)
    bad = []
    if int(n_records) != n:
        bad.append(f"kernel {k}: n_records {n_records} != {n}")
    for p, d in expected(cfg, k, roles_of(k, P)).items():
        for f, v in d.items():
            if int(keys[f][p]) != v:
                bad.append(f"kernel {k} pc {p} {f}: {int(keys[f][p])} != {v}")
    tot = int(np.sum(keys["n_ld"][:P])) + int(np.sum(keys["n_st"][:P]))
    if tot != n:
        bad.append(f"kernel {k}: per-PC counts sum {tot} != {n}")
    return bad
