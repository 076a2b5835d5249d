"""the value flow graph (Defs 5.1-5.3).

Oracle pins (C18-C20): the Figure 3 program as the text walks it (edges
1->3, 2->4, 3->5, 4->6, 5->7 (read), 6->7 (write)) and its vertex slice on vertex 6
(Fig. 3d: the inputs and outputs of vertex 6 only), host copies as source / sink
edges, merged invocations of one call path, the important-graph
thresholds (Def 5.3).  libve's graph builder is host code (no device): its parity
with the oracle runs here on random logs, CPU only."""
import numpy as np
import pytest

from oracle import oracle as O

R, W = 1, 2
DEV, ALLOC, H2D, D2H = 0, 1, 2, 3
HOST = O.HOST_VERTEX


def log(rows):
    """rows: (seq, vertex, object, mode, kind, bytes)"""
    a = np.zeros(len(rows), dtype=O.ACCESS_DTYPE)
    for i, (seq, v, k, m, kind, b) in enumerate(rows):
        a[i] = (seq, b, v, k, m, kind)
    return a


def E(edges):
    return sorted((int(e["src"]), int(e["dst"]), int(e["object"]), int(e["label"])) for e in edges)


N = 1 << 20
A, B = 0, 1
FIG3 = log([(1, 1, A, W, ALLOC, 4 * N), (2, 2, B, W, ALLOC, 4 * N),                 # cudaMalloc A_dev, B_dev
            (3, 3, A, W, DEV, 4 * N), (4, 4, B, W, DEV, 4 * N),                     # cudaMemset A_dev, B_dev
            (5, 5, A, W, DEV, 4 * N), (6, 6, B, W, DEV, 4 * N),                     # kernels writing zeros
            (7, 7, A, R, DEV, 4 * N), (7, 7, B, W, DEV, 4 * N)])                    # reads A_dev, writes B_dev


def test_figure3_edges():
    e, v = O.vfg_build(FIG3)
    assert E(e) == [(1, 3, A, W), (2, 4, B, W), (3, 5, A, W), (4, 6, B, W), (5, 7, A, R), (6, 7, B, W)]
    assert [int(x["vertex"]) for x in v] == list(range(1, 8)) and all(int(x["invocations"]) == 1 for x in v)


def test_figure3_slice_of_vertex6():
    e, v = O.vfg_build(FIG3)
    se, sv = O.vfg_slice(e, v, 6)
    assert E(se) == [(2, 4, B, W), (4, 6, B, W), (6, 7, B, W)]
    assert [int(x["vertex"]) for x in sv] == [2, 4, 6, 7]


def test_host_copies_and_merged_invocations():
    rows = [(1, 1, A, W, ALLOC, 64), (2, 2, A, W, H2D, 64), (3, 3, A, R, DEV, 64), (4, 4, A, R, D2H, 64)]
    rows += [(5 + i, 5, A, R | W, DEV, 32) for i in range(3)]                      # one call path, 3 launches
    e, v = O.vfg_build(log(rows))
    got = {(int(x["src"]), int(x["dst"]), int(x["object"])): (int(x["label"]), int(x["bytes"]), int(x["count"]))
           for x in e}
    assert got == {(1, 2, A): (W, 64, 1), (HOST, 2, A): (W, 64, 1), (2, 3, A): (R, 64, 1), (2, 4, A): (R, 64, 1),
                   (4, HOST, A): (R, 64, 1), (2, 5, A): (R | W, 32, 1), (5, 5, A): (R | W, 64, 2)}
    assert {int(x["vertex"]): int(x["invocations"]) for x in v} == {1: 1, 2: 1, 3: 1, 4: 1, 5: 3}
    ie, iv = O.vfg_important(e, v, 64, 2)           # edges of >= 64 bytes; vertices on them or invoked >= 2 times
    assert len(ie) == 6 and sorted(int(x["vertex"]) for x in iv) == [1, 2, 3, 4, 5]
    ie, iv = O.vfg_important(e, v, 65, 3)
    assert len(ie) == 0 and [int(x["vertex"]) for x in iv] == [5]


def test_access_before_allocation_rejected():
    with pytest.raises(ValueError):
        O.vfg_build(log([(1, 1, A, R, DEV, 4)]))


def _random_log(seed):
    rng = np.random.default_rng(seed)
    rows, seq, allocated = [], 0, []
    for _ in range(int(rng.integers(5, 60))):
        seq += 1
        v = int(rng.integers(0, 12))                                   # call paths repeat
        if not allocated or rng.random() < 0.15:
            k = len(allocated)
            allocated.append(k)
            rows.append((seq, 100 + k, k, W, ALLOC, 8))
            continue
        kind = int(rng.choice([DEV, DEV, DEV, H2D, D2H]))
        for k in set(int(x) for x in rng.choice(allocated, int(rng.integers(1, 3)))):
            rows.append((seq, v, k, int(rng.integers(1, 4)), kind, int(rng.integers(1, 100))))
    return log(rows)


@pytest.mark.parametrize("seed", range(10))
def test_libve_graph_matches_oracle(seed):
    """libve's host-side builder / slice / important graph against C18-C20 (no device needed)."""
    from paper_conf_asplos_zhouhmm022_b200 import ve
    lg = _random_log(seed)
    g = ve.ValueFlowGraph.build(lg)
    oe, ov = O.vfg_build(lg)
    assert g.edges.tobytes() == oe.tobytes() and g.vertices.tobytes() == ov.tobytes()
    for vtx in [int(x["vertex"]) for x in ov][:6]:
        s = g.slice(vtx)
        se, sv = O.vfg_slice(oe, ov, vtx)
        assert s.edges.tobytes() == se.tobytes() and s.vertices.tobytes() == sv.tobytes()
    for eb, vi in ((1, 1), (50, 2), (200, 5)):
        i = g.important(eb, vi)
        ie, iv = O.vfg_important(oe, ov, eb, vi)
        assert i.edges.tobytes() == ie.tobytes() and i.vertices.tobytes() == iv.tobytes()


def test_libve_figure3():
    from paper_conf_asplos_zhouhmm022_b200 import ve
    g = ve.ValueFlowGraph.build(FIG3)
    assert E(g.edges) == [(1, 3, A, W), (2, 4, B, W), (3, 5, A, W), (4, 6, B, W), (5, 7, A, R), (6, 7, B, W)]
    assert E(g.slice(6).edges) == [(2, 4, B, W), (4, 6, B, W), (6, 7, B, W)]
    with pytest.raises(ve.VeError):
        ve.ValueFlowGraph.build(log([(2, 1, A, W, ALLOC, 4), (1, 2, A, R, DEV, 4)]))   # not in program order


def test_cfg5_api_log_graph():
    """f4 at the paper's scale (LAMMPS: 660 vertices pruned to 132, Def 5.3): the value flow graph
    of cfg5's 4000-kernel API log (1000 objects, 64 kernel call paths) -- libve's builder, slice and
    important graph against the oracle, and the invariants of the log's construction: one vertex per
    call path, invocations = launches per path, every object's first edge leaves its allocation."""
    from paper_conf_asplos_zhouhmm022_b200 import ve
    from tests import workloads as WL
    lg = WL.cfg5_api_log()
    g = ve.ValueFlowGraph.build(lg)
    oe, ov = O.vfg_build(lg)
    assert g.edges.tobytes() == oe.tobytes() and g.vertices.tobytes() == ov.tobytes()
    inv = {int(x["vertex"]): int(x["invocations"]) for x in ov}
    launches = {}
    for r in lg:
        if int(r["kind"]) == DEV:
            launches.setdefault(int(r["vertex"]), set()).add(int(r["seq"]))
    for v, seqs in launches.items():
        assert inv[v] == len(seqs)
    assert sum(1 for v in inv if 100 <= v < 164) == 64
    # Def 5.3: keep edges of >= 16 MiB and vertices invoked >= 70 times; the pruned graph is smaller
    ie, iv = O.vfg_important(oe, ov, 16 << 20, 70)
    gi = g.important(16 << 20, 70)
    assert gi.edges.tobytes() == ie.tobytes() and gi.vertices.tobytes() == iv.tobytes()
    assert 0 < len(ie) < len(oe) // 10 and len(iv) <= len(ov)
    v0 = int(ov[len(ov) // 2]["vertex"])
    se, sv = O.vfg_slice(oe, ov, v0)
    s = g.slice(v0)
    assert s.edges.tobytes() == se.tobytes() and s.vertices.tobytes() == sv.tobytes()
