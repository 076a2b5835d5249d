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
CFG5_SEED, CFG5_N, CFG5_UNIT = 5, 1000, 8 << 20     # 1000 objects, 4 sizes of 8-32 MiB: ~19.5 GiB


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
