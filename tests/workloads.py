"""Seeded workloads shared by the GPU parity tests, smoke() and bench.py: the
same generator inputs laid out for the oracle (host) and for libve (device).
Input plumbing only -- no analysis arithmetic."""
import numpy as np

from gen import vegen as G


def host_objects(cfg, epoch, seed):
    objs = []
    for i, o in enumerate(G.objects(cfg, epoch)):
        d = dict(o)
        d["pre"] = G.snapshot_host(cfg, epoch, seed, i, 0) if o["has_pre"] else None
        d["post"] = G.snapshot_host(cfg, epoch, seed, i, 1) if o["has_post"] else None
        objs.append(d)
    return objs


def device_objects(host_objs, device="cuda"):
    import torch
    out = []
    for o in host_objs:
        d = {k: o[k] for k in ("base", "size", "id", "elem_width")}
        d["pre"] = torch.from_numpy(o["pre"]).to(device) if o.get("pre") is not None else None
        d["post"] = torch.from_numpy(o["post"]).to(device) if o.get("post") is not None else None
        out.append(d)
    return out


def device_records(recs, device="cuda"):
    import torch
    return torch.from_numpy(np.ascontiguousarray(recs).view(np.uint8)).to(device)


# ---- cfg5 duplicate-object scan (dedup half) ------------------------------
# 1000 objects; unit 0 = the recipe's sizing: 50 log-uniform size classes over [64 KiB, 512 MiB], rescaled
# to 20 GiB in total (gen/ve_gen_core.h veg_dedup_size)
CFG5_SEED, CFG5_N, CFG5_UNIT = 5, 1000, 0


def cfg5_dedup_objects(n=CFG5_N, unit=CFG5_UNIT, seed=CFG5_SEED):
    """Object table of the cfg5 duplicate scan (generator metadata: size, content class, copy source)."""
    return [G.dedup_object(seed, i, unit) for i in range(n)]


def cfg5_expected_groups(objs):
    """Closed form of the duplicate classes from the generator's construction (not from any analysis):
    class 0 = zeros, 3 = random (own content), 1 = exact copy of src, 2 = copy of src with one bit
    flipped (a content of its own).  group_of[i] = min id with the same content."""
    key = {}
    for o in objs:
        c, s = o["cls"], o["src"]
        if c == 0 or (c == 1 and objs[s]["cls"] == 0):
            key[o["id"]] = ("z", o["size"])
        elif c == 3:
            key[o["id"]] = ("r", o["id"])
        elif c == 1:
            key[o["id"]] = ("r", s)
        else:
            key[o["id"]] = ("f", o["id"])
    first = {}
    for o in objs:
        first.setdefault(key[o["id"]], o["id"])
    return [first[key[o["id"]]] for o in objs]


# ---- cfg5 API-event log (the value flow graph of the 4000-kernel application) ----
def cfg5_api_log(seed=CFG5_SEED, n_obj=CFG5_N, kernels=4000, sites=64):
    """The API-event log of BASELINE configs[4] as the value flow graph sees it (Def 5.1):
    the 1000 objects of the duplicate-scan set are allocated (7 allocation call sites) and 30% of them
    filled from the host (5 copy sites); then 4000 kernel launches from `sites` call paths (P:L275:
    invocations of one call path are one vertex), kernel k touching the veg_c5_nobj(k) objects its
    geometry gives (1..4), drawn from the 1000 by a seeded generator, each read (60%), written (15%)
    or both (25%), with the bytes its records cover; at the end 10% of the objects are copied back.
    Input plumbing only: the rows of an ACCESS_DTYPE log (seq, bytes, vertex, object, mode, kind)."""
    rng = np.random.default_rng(seed)
    objs = cfg5_dedup_objects(n_obj)
    rows, seq = [], 0
    R, Wr, DEV, ALLOC, H2D, D2H = 1, 2, 0, 1, 2, 3
    for o in objs:
        seq += 1
        rows.append((seq, o["size"], 1 + o["id"] % 7, o["id"], Wr, ALLOC))
    for o in objs:
        if rng.random() < 0.3:
            seq += 1
            rows.append((seq, o["size"], 10 + o["id"] % 5, o["id"], Wr, H2D))
    cfg = G.scaled(G.CFG5, 0)
    for k in range(kernels):
        seq += 1
        inf = G.info(cfg, k)
        nobj, nrec = inf["n_obj"], inf["n_records"]
        for j in sorted(set(int(x) for x in rng.choice(n_obj, nobj, replace=False))):
            u = rng.random()
            mode = R if u < 0.6 else (Wr if u < 0.75 else R | Wr)
            rows.append((seq, min(4 * nrec // nobj, objs[j]["size"]), 100 + k % sites, j, mode, DEV))
    for o in objs:
        if rng.random() < 0.1:
            seq += 1
            rows.append((seq, o["size"], 20, o["id"], R, D2H))
    a = np.zeros(len(rows), dtype=[("seq", "<u8"), ("bytes", "<u8"), ("vertex", "<u4"), ("object", "<u4"),
                                   ("mode", "<u4"), ("kind", "<u4")])
    for i, r in enumerate(rows):
        a[i] = r
    return a
