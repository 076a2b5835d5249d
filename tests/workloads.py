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
