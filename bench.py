"""bench.py -- value-trace analysis throughput on B200 (BASELINE.json metric).

One step = one pass of the whole hot path over the N=1
workload, BASELINE.json configs[1] (cfg2, Darknet YOLOv4 conv layer, 231.6 M
records, 5.56 GB of trace):
  epoch 0 (fill_ongpu):  set_objects -> analyze 5.9 M records -> snapshot diff(output) -> report
  epoch 1 (gemm beta=1): set_objects -> analyze 225.6 M records -> snapshot diff(output) -> report
  duplicate scan over {weights, workspace, output, x_gpu}.
Inputs are generated on the device before timing (5.56 GB > 126 MB L2, so no
flush is needed).  With --gpus N (torchrun) each rank analyzes its contiguous
1/N of every epoch and the ranks merge over NCCL (strong scaling).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl reference]
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "value-trace records/sec (trace GB/s vs HBM peak) at 1/2/4/8 B200"
UNIT = "records/s"
REC_BYTES = 24
PEAKS = os.path.join(ROOT, "MEASURED_PEAKS.json")


def hbm_peak():
    try:
        with open(PEAKS) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class Clocks:
    """nvidia-smi sampler running during the timed region (B200_PROFILING.md clocks line)."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for ln in self.proc.stdout:
            self.lines.append(ln.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        self.t.join(timeout=2)
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 6:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for nm, v in zip(names, parts[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------------------- workload
class Workload:
    """cfg2 on the device: records of this rank's share of each epoch + snapshots."""

    def __init__(self, rank, world, device):
        import torch
        from gen import vegen as G
        self.G, self.torch = G, torch
        self.seed = G.SEEDS[G.CFG2]
        self.device = device
        self.epochs = []
        stream = torch.cuda.current_stream().cuda_stream
        self.total_records = 0
        for ep in (0, 1):
            inf = G.info(G.CFG2, ep)
            n = inf["n_records"]
            self.total_records += n
            lo, hi = n * rank // world, n * (rank + 1) // world   # = ve.rank_chunk
            recs = torch.empty((hi - lo) * REC_BYTES, dtype=torch.uint8, device=device)
            G.records_device(G.CFG2, ep, self.seed, lo, hi - lo, recs.data_ptr(), stream)
            objs = []
            for i, o in enumerate(G.objects(G.CFG2, ep)):
                pre = torch.empty(o["size"], dtype=torch.uint8, device=device)
                post = torch.empty(o["size"], dtype=torch.uint8, device=device)
                G.snapshot_device(G.CFG2, ep, self.seed, i, 0, pre.data_ptr(), stream)
                G.snapshot_device(G.CFG2, ep, self.seed, i, 1, post.data_ptr(), stream)
                objs.append({"base": o["base"], "size": o["size"], "id": o["id"], "elem_width": o["elem_width"],
                             "pre": pre, "post": post})
            self.epochs.append({"n_pcs": inf["n_pcs"], "lo": lo, "n": hi - lo, "recs": recs, "objs": objs,
                                "n_total": n})
        torch.cuda.synchronize()
        self.trace_bytes = self.total_records * REC_BYTES
        # algorithmic bytes: 24 B per record + one read of every pre element referenced
        # with eq_pre defined (U).  Epoch 0 touches output (5,914,624 elements); epoch 1 touches
        # weights, workspace and output in full.
        u0 = 5914624
        u1 = 294912 + 6653952 + 5914624
        self.alg_bytes_epoch = [G.info(G.CFG2, 0)["n_records"] * REC_BYTES + 4 * u0,
                                G.info(G.CFG2, 1)["n_records"] * REC_BYTES + 4 * u1]

    def dedup_objs(self):
        o = self.epochs[1]["objs"]
        return [{"base": x["base"], "size": x["size"], "id": x["id"], "elem_width": 4, "pre": None,
                 "post": x["post"]} for x in o] + \
               [{"base": 0x7f9000000000, "size": o[2]["size"], "id": 4, "elem_width": 4, "pre": None,
                 "post": self.epochs[0]["objs"][2]["post"]}]


def run_step(ctx, wl, tstream, ev_pairs=None, comm=None):
    """One pass of the hot path; returns the reports (for the parity spot check) and dedup groups."""
    stream = tstream.cuda_stream
    reps = []
    for ep, e in enumerate(wl.epochs):
        ctx.set_objects(e["objs"])
        if ev_pairs is not None:
            ev_pairs[ep][0].record(tstream)
        ctx.analyze_records(e["recs"], e["n"], stream=stream)
        if ev_pairs is not None:
            ev_pairs[ep][1].record(tstream)
        if comm is not None:
            ctx.merge(comm=comm, stream=stream)
        ctx.snapshot_diff(2, stream=stream)
        reps.append(ctx.report())
    groups = ctx.object_dedup(wl.dedup_objs(), stream=stream)
    return reps, groups


# ----------------------------------------------------------------------------- CPU oracle arm
def oracle_sample(n_sample, seed_offset=0):
    """Bounded sample of the same workload for the oracle: the first n_sample records of the gemm
    epoch (A/B/C interleaved exactly as in the full trace) with full snapshots."""
    from gen import vegen as G
    from oracle import oracle as O
    seed = G.SEEDS[G.CFG2]
    recs = G.records_host(G.CFG2, 1, seed, seed_offset, n_sample)
    objs = []
    for i, o in enumerate(G.objects(G.CFG2, 1)):
        d = dict(o)
        d["pre"] = G.snapshot_host(G.CFG2, 1, seed, i, 0)
        d["post"] = G.snapshot_host(G.CFG2, 1, seed, i, 1)
        objs.append(d)
    return O, O.make_config(G.info(G.CFG2, 1)["n_pcs"]), objs, recs


def time_oracle(n_sample):
    O, cfg, objs, recs = oracle_sample(n_sample)
    t = time.perf_counter()
    O.analyze(cfg, objs, recs)
    dt = time.perf_counter() - t
    return n_sample / dt, dt


def reference_arm(args, rank, world):
    """--impl reference: the CPU oracle, as it stands, on the host (rank 0 only)."""
    if rank != 0:
        return
    n_sample = args.ref_sample
    O, cfg, objs, recs = oracle_sample(n_sample)
    for _ in range(args.warmup):
        O.analyze(cfg, objs, recs[: max(1, n_sample // 16)])
    times = []
    for _ in range(args.steps):
        t = time.perf_counter()
        O.analyze(cfg, objs, recs)
        times.append(time.perf_counter() - t)
    total = sum(times)
    v = n_sample * args.steps / total
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * total / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic (seeded counter-based generator)",
            "config": workload_config(sample=n_sample),
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"first {n_sample} records of the cfg2 gemm epoch, full snapshots, per step"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def workload_config(sample=None, world=1):
    from gen import vegen as G
    n = G.info(G.CFG2, 0)["n_records"] + G.info(G.CFG2, 1)["n_records"]
    c = {"workload": "cfg2: Darknet YOLOv4 conv layer trace (fill_ongpu + gemm beta=1; M=256 K=1152 N=5776 batch 4)",
         "records": n, "trace_bytes": n * REC_BYTES, "pcs": 5, "objects": 4,
         "l2": "inputs larger than L2 (5.56 GB trace vs 126 MB), no flush",
         "parallelism": f"dp{world} (record chunks + NCCL merge)" if world > 1 else "single GPU"}
    if sample is not None:
        c["sample_records"] = sample
    return c


# ----------------------------------------------------------------------------- GPU arm
def max_over_ranks(ms, device="cuda"):
    """The slowest rank's device time (the job's time under strong scaling)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([float(ms)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--ref-sample", type=int, default=4_000_000)
    ap.add_argument("--cpu-sample", type=int, default=16_000_000)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-f1", action="store_true")
    ap.add_argument("--no-cfg5", action="store_true")
    ap.add_argument("--no-cfg34", action="store_true")
    args = ap.parse_args()

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return reference_arm(args, rank, world)

    import torch
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=dev)
    from paper_conf_asplos_zhouhmm022_b200 import ve

    wl = Workload(rank, world, dev)
    # hist_capacity >= 2x the distinct (pc, object, value) entries of an epoch:
    # cfg2's gemm epoch has 1,274,116 (scripts/cfg2_ndistinct.py), so 2^22 slots (30% load)
    ctx = ve.Context(n_pcs=5, max_objects=8, hist_capacity=int(os.environ.get("VE_BENCH_HCAP", 1 << 22)),
                     device=local)
    comm = None
    if world > 1:
        comm = ve.nccl_comm_from_torch(rank, world)
    stream = torch.cuda.current_stream()

    for _ in range(args.warmup):
        run_step(ctx, wl, stream, comm=comm)
    torch.cuda.synchronize()

    evs = [[[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(2)] for _ in range(args.steps)]
    clk = Clocks(local)
    launches0 = ve.kernel_launches()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    clk.start()
    time.sleep(0.3)
    start.record(stream)
    for k in range(args.steps):
        reps, groups = run_step(ctx, wl, stream, ev_pairs=evs[k], comm=comm)
    end.record(stream)
    torch.cuda.synchronize()
    clocks = clk.stop()
    launches = ve.kernel_launches() - launches0
    ms = start.elapsed_time(end)
    if world > 1:
        ms = max_over_ranks(ms, device=dev)
    ms_step = ms / args.steps
    value = wl.total_records / (ms_step / 1e3)

    # roofline of the dominant kernel (k_analyze): algorithmic bytes / CUDA-event duration per launch
    an_ms = [[evs[k][ep][0].elapsed_time(evs[k][ep][1]) for ep in (0, 1)] for k in range(args.steps)]
    alg = [b / world for b in wl.alg_bytes_epoch]
    ep1_ms = statistics.mean(a[1] for a in an_ms)
    achieved = alg[1] / (ep1_ms / 1e3) / 1e9
    peak, peak_src = hbm_peak()
    traffic = None
    prof = os.path.join(ROOT, "profiles", "k_analyze_traffic.json")
    if os.path.exists(prof):
        try:
            traffic = json.load(open(prof)).get("dram_bytes_per_launch")
        except Exception:
            traffic = None

    # parity spot check on the full-size run: properties that hold at any size (closed forms of cfg2)
    k0, k1 = reps[0].keys, reps[1].keys
    spot = {
        "fill_redundant_stores": int(k0["n_st_eq_pre"][0]) == wl.epochs[0]["n_total"],
        "c_load_single_zero": bool(k1["single_zero"][3]) and int(k1["n_ld_eq_pre"][3]) == 5914624,
        "a_loads": int(k1["n_ld"][1]) == 107347968, "b_loads": int(k1["n_ld"][2]) == 106463232,
        "dedup_output_xgpu": int(groups[4]) == 3 and int(groups[3]) == 3,
    }

    f1 = None
    if rank == 0 and world == 1 and not args.no_f1:       # single-GPU legs: not under torchrun
        f1 = measure_next_rows(ve, ctx, wl, stream, peak)

    dd5 = r5 = None
    if rank == 0 and world == 1 and not args.no_cfg5:
        dd5 = measure_cfg5_dedup(ve, ctx, stream, peak)
        r5 = measure_cfg5_records(ve, stream, peak)
    c34 = None
    if rank == 0 and world == 1 and not args.no_cfg34:
        c34 = measure_other_configs(ve, stream, peak)

    e2e = None
    if not args.no_e2e and rank == 0 and world == 1:
        e2e = measure_e2e(ve, ctx, wl, stream, max(1, min(args.steps, 3)))

    cpu = None
    if not args.no_cpu and rank == 0 and world == 1:
        rate, dt = time_oracle(args.cpu_sample)
        cpu = {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"first {args.cpu_sample} records of the cfg2 gemm epoch (A/B/C interleaved), full snapshots;"
                         f" {dt:.1f} s single-threaded"}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": "u64", "data": "synthetic (seeded counter-based generator, cfg2 recipe)",
                "config": workload_config(world=world),
                "trace_gbs": value * REC_BYTES / 1e9,
                "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                             "frac": achieved / peak, "traffic": traffic, "kernel": "k_analyze (gemm epoch launch)",
                             "peak_source": peak_src, "ms_per_launch": ep1_ms,
                             "alg_bytes_per_launch": alg[1]},
                "analyze_ms_per_step": [round(statistics.mean(a[i] for a in an_ms), 4) for i in (0, 1)],
                "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches, "clocks": clocks,
                "next_rows": f1, "cfg5_dedup": dd5, "cfg5_records": r5, "cfg3_cfg4": c34,
                "parity_spot_check": spot}
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()


def measure_next_rows(ve, ctx, wl, stream, peak, reps=3):
    """SURVEY 8(f) rows, measured outside the step on this rank's cfg2 gemm-epoch records (CUDA events
    around each synchronizing call, median of `reps`):
      f1 ve_record_intervals (warp compaction, radix sort, merge scans),
      f2 ve_approx_topk on the ctx's gemm-epoch histogram (re-keyed by truncated value),
      f3 ve_temporal_loads (ordered load compaction, radix sort by address, neighbour judging),
      f2 ve_dyadic_fit (three streaming passes over the records: algorithmic bytes 3 x 24 B per record)."""
    import torch
    e = wl.epochs[1]
    n = e["n"]
    sp = stream.cuda_stream

    def timed(fn):
        fn()                                    # warm-up (workspace pool)
        ts, r = [], None
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            a.record(stream)
            r = fn()
            b.record(stream)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return statistics.median(ts), r

    out = torch.empty(n * 16, dtype=torch.uint8, device=wl.device)
    ms1, k = timed(lambda: ctx.record_intervals(e["recs"], n, out, stream=sp))
    del out
    ctx.set_objects(e["objs"])
    ctx.analyze_records(e["recs"], n, stream=sp)
    ms2, (nd, _top) = timed(lambda: ctx.approx_topk(stream=sp))
    ms3, tl = timed(lambda: ctx.temporal_loads(e["recs"], n, stream=sp))
    ms4, dy = timed(lambda: ctx.dyadic_fit(e["recs"], n, stream=sp))
    gbs = lambda ms: n * REC_BYTES / (ms / 1e3) / 1e9
    return {
        "note": "SURVEY 8(f) rows, not part of the step; each call synchronizes (count read-backs) inside its "
                "timed region",
        "f1_record_intervals": {"records": n, "ms": ms1, "records_per_s": n / (ms1 / 1e3), "trace_gbs": gbs(ms1),
                                "frac_of_hbm_peak": gbs(ms1) / peak, "merged_intervals": k},
        "f2_approx_topk": {"ms": ms2, "keys_with_approx_histogram": int((nd > 0).sum()),
                           "approx_distinct_total": int(nd.sum())},
        "f3_temporal_loads": {"records": n, "ms": ms3, "records_per_s": n / (ms3 / 1e3), "trace_gbs": gbs(ms3),
                              "frac_of_hbm_peak": gbs(ms3) / peak, "temporal_loads_pc": [int(x) for x in tl[:5, 0]],
                              "closed_form_ok": bool(int(tl[1, 1]) == 363 * 256 * 1152
                                                     and int(tl[2, 1]) == 15 * 1152 * 5776)},
        "f2_dyadic_fit": {"records": n, "ms": ms4, "records_per_s": n / (ms4 / 1e3),
                          "alg_gbs": 3 * gbs(ms4), "frac_of_hbm_peak": 3 * gbs(ms4) / peak,
                          "states": [int(x) for x in np.bincount(dy["state"], minlength=4)]},
    }


def measure_other_configs(ve, stream, peak):
    """BASELINE configs[2] (cfg3, PyTorch op mix: 4 iterations x 264 M records) and configs[3] (cfg4, f64
    stencils: 1.07 G + 0.94 G records), full size, outside the step: per epoch the records and snapshots
    are generated on the device (untimed), then set_objects + ve_analyze_records + ve_report are timed with
    CUDA events.  Parity at full size: the recipe's closed forms (tests/cfg34.py)."""
    import torch
    from gen import vegen as G
    from tests import cfg34
    sp = stream.cuda_stream
    out = {}
    plans = [("cfg3", G.scaled(G.CFG3, 0), [(0, 3), (0, 4), (0, 5), (0, 6)], 1 << 25),
             ("cfg4", G.scaled(G.CFG4, 0), [(0, 4), (1, 4)], 1 << 22)]
    for name, cfg, runs, hcap in plans:
        tot_n, tot_ms, ok = 0, 0.0, True
        for epoch, seed in runs:
            inf = G.info(cfg, epoch)
            n = inf["n_records"]
            dobjs = []
            for i, o in enumerate(G.objects(cfg, epoch)):
                d = {k: o[k] for k in ("base", "size", "id", "elem_width")}
                for side in ("pre", "post"):
                    t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
                    G.snapshot_device(cfg, epoch, seed, i, side == "post", t.data_ptr(), sp)
                    d[side] = t
                dobjs.append(d)
            recs = torch.empty(n * REC_BYTES, dtype=torch.uint8, device="cuda")
            G.records_device(cfg, epoch, seed, 0, n, recs.data_ptr(), sp)
            ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=len(dobjs), hist_capacity=hcap)
            for rep_i in range(2):           # pass 0 warms the context (allocations, pools), pass 1 is timed
                torch.cuda.synchronize()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                ctx.set_objects(dobjs)
                ctx.analyze_records(recs, n, stream=sp)
                rep = ctx.report()
                b.record(stream)
                torch.cuda.synchronize()
            tot_ms += a.elapsed_time(b)
            tot_n += n
            if seed == runs[0][1] and epoch in (0, 1):
                k = {f: rep.keys[f] for f in rep.keys.dtype.names}
                k["top_bits"], k["top_count"] = rep.topk["bits"], rep.topk["count"]
                bad = (cfg34.check_cfg3(k, int(rep.globals["n_records"]), 0, rep.objects) if name == "cfg3" else
                       cfg34.check_cfg4(k, int(rep.globals["n_records"]), 0, epoch, rep.objects))
                ok = ok and not bad
            ctx.close()
            del dobjs, recs
            torch.cuda.empty_cache()
        gbs = tot_n * REC_BYTES / (tot_ms / 1e3) / 1e9
        out[name] = {"records": tot_n, "ms": tot_ms, "records_per_s": tot_n / (tot_ms / 1e3), "trace_gbs": gbs,
                     "trace_frac_of_hbm_peak": gbs / peak, "closed_forms_ok": ok,
                     "timed": "set_objects + analyze + report per epoch (no diff / dedup), second pass on a warm "
                              "context"}
    return out


def measure_cfg5_dedup(ve, ctx, stream, peak, reps=3):
    """BASELINE configs[4] (cfg5), duplicate-object half: ve_object_dedup over 1000 objects / ~19.7 GiB of
    post snapshots generated on the device (untimed); CUDA events around the (synchronizing) call.
    Algorithmic bytes: every byte hashed once + 2 x size per non-representative duplicate."""
    import torch
    from gen import vegen as G
    from tests import workloads as W
    objs = W.cfg5_dedup_objects()
    sp = stream.cuda_stream
    dobjs = []
    for o in objs:
        t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
        G.dedup_device(W.CFG5_SEED, o["id"], W.CFG5_UNIT, t.data_ptr(), sp)
        dobjs.append(dict(o, pre=None, post=t))
    torch.cuda.synchronize()
    want = W.cfg5_expected_groups(objs)
    g = ctx.object_dedup(dobjs, stream=sp)                     # warm-up
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(stream)
        g = ctx.object_dedup(dobjs, stream=sp)
        b.record(stream)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ms = statistics.median(ts)
    total = sum(o["size"] for o in objs)
    dup = sum(o["size"] for o, w in zip(objs, want) if w != o["id"])
    alg = total + 2 * dup
    del dobjs
    torch.cuda.empty_cache()
    return {"workload": "cfg5 duplicate-object scan: 1000 objects, 4 sizes (8-32 MiB), 30% zero / 10% copies / "
                        "5% one-bit flips / 55% random", "objects": len(objs), "bytes": total, "ms": ms,
            "alg_bytes": alg, "alg_gbs": alg / (ms / 1e3) / 1e9, "frac_of_hbm_peak": alg / (ms / 1e3) / 1e9 / peak,
            "groups": len(set(want)), "parity_closed_form": [int(x) for x in g] == want}


def measure_cfg5_records(ve, stream, peak):
    """BASELINE configs[4] (cfg5), records half: 4000 independent kernels, 10^9 records in total (4..64 PCs,
    1..4 objects, 2,987 .. 1,676,166 records each; gen/ve_gen_core.h veg_cfg5_record).  All records and
    snapshots are generated on the device first (untimed, 24 GB + 2 x 4 GB); the timed region is the
    per-kernel analysis a user runs -- ve_set_objects + ve_analyze_records + ve_report for every kernel
    on ONE context -- bracketed by CUDA events; events around each ve_analyze_records give the share of
    the analysis kernels.  Parity at full size: the recipe's closed forms (tests/cfg5k.py) on every 50th
    kernel (kernel-by-kernel oracle parity is tests/test_gpu_cfg5.py)."""
    import torch
    from gen import vegen as G
    from tests import cfg5k
    sp = stream.cuda_stream
    cfg, seed, K = G.scaled(G.CFG5, 0), 5, 4000
    infos = [G.info(cfg, k) for k in range(K)]
    n_tot = sum(i["n_records"] for i in infos)
    recs = torch.empty(n_tot * REC_BYTES, dtype=torch.uint8, device="cuda")
    objs_of = [G.objects(cfg, k) for k in range(K)]
    snap_tot = sum(o["size"] for objs in objs_of for o in objs)
    snaps = torch.empty(2 * snap_tot, dtype=torch.uint8, device="cuda")
    r0, s0, plan = 0, 0, []
    for k in range(K):
        n = infos[k]["n_records"]
        G.records_device(cfg, k, seed, 0, n, recs.data_ptr() + r0 * REC_BYTES, sp)
        dobjs = []
        for i, o in enumerate(objs_of[k]):
            d = {f: o[f] for f in ("base", "size", "id", "elem_width")}
            for side in ("pre", "post"):
                t = snaps[s0:s0 + o["size"]]
                s0 += o["size"]
                G.snapshot_device(cfg, k, seed, i, side == "post", t.data_ptr(), sp)
                d[side] = t
            dobjs.append(d)
        plan.append((recs[r0 * REC_BYTES:(r0 + n) * REC_BYTES], n, dobjs))
        r0 += n
    ctx = ve.Context(n_pcs=64, max_objects=4, hist_capacity=1 << 23)
    for buf, n, dobjs in plan[:8]:                                 # warm the context (untimed)
        ctx.set_objects(dobjs)
        ctx.analyze_records(buf, n, stream=sp)
        ctx.report().close()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    bad, checked = [], 0
    a.record(stream)
    for k, (buf, n, dobjs) in enumerate(plan):
        ctx.set_objects(dobjs)
        ev[k][0].record(stream)
        ctx.analyze_records(buf, n, stream=sp)
        ev[k][1].record(stream)
        rep = ctx.report()
        if k % 50 == 0:
            keys = {f: rep.keys[f].copy() for f in ("n_ld", "n_st", "n_ld_eq_pre", "n_st_eq_pre", "raw_min",
                                                     "raw_max", "single_zero", "single_value")}
            plan[k] = (buf, n, dobjs, keys, int(rep.globals["n_records"]))
        rep.close()
    b.record(stream)
    torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    an_ms = sum(x.elapsed_time(y) for x, y in ev)
    for k in range(0, K, 50):
        bad += cfg5k.check_cfg5_kernel(plan[k][3], plan[k][4], cfg, k)
        checked += 1
    ctx.close()
    del plan, recs, snaps
    torch.cuda.empty_cache()
    gbs = n_tot * REC_BYTES / (ms / 1e3) / 1e9
    return {"workload": "cfg5 records: 4000 kernels, 4-64 PCs with cfg1 roles, 1-4 objects, 10^9 records",
            "kernels": K, "records": n_tot, "snapshot_bytes": 2 * snap_tot, "ms": ms,
            "records_per_s": n_tot / (ms / 1e3), "trace_gbs": gbs, "trace_frac_of_hbm_peak": gbs / peak,
            "analyze_ms": an_ms, "analyze_records_per_s": n_tot / (an_ms / 1e3),
            "per_kernel_overhead_ms": (ms - an_ms) / K, "closed_forms_kernels_checked": checked,
            "closed_forms_ok": not bad, "closed_form_mismatches": bad[:5],
            "timed": "set_objects + analyze + report per kernel on one context, CUDA events around the loop"}


def measure_e2e(ve, ctx, wl, stream, steps):
    """Same metric through the public API from pinned HOST buffers: H2D of every input (records and
    snapshots) and D2H of the reports are inside the timed region."""
    import torch
    host = []
    h2d = 0
    for e in wl.epochs:
        hr = torch.empty(e["recs"].numel(), dtype=torch.uint8, pin_memory=True)
        hr.copy_(e["recs"])
        snaps = [(torch.empty(o["size"], dtype=torch.uint8, pin_memory=True).copy_(o["pre"]),
                  torch.empty(o["size"], dtype=torch.uint8, pin_memory=True).copy_(o["post"])) for o in e["objs"]]
        host.append((hr, snaps))
        h2d += hr.numel() + sum(2 * o["size"] for o in e["objs"])
    torch.cuda.synchronize()
    d2h = 0

    def step():
        nonlocal d2h
        d2h = 0
        for ep, e in enumerate(wl.epochs):
            hr, snaps = host[ep]
            for o, (hp, hq) in zip(e["objs"], snaps):
                o["pre"].copy_(hp, non_blocking=True)
                o["post"].copy_(hq, non_blocking=True)
            ctx.set_objects(e["objs"])
            ctx.analyze_records_host(hr, e["n"], stream=stream.cuda_stream)
            ctx.snapshot_diff(2, stream=stream.cuda_stream)
            rep = ctx.report()
            d2h += rep.keys.nbytes + rep.topk.nbytes + rep.objects.nbytes + 32 + 48
        ctx.object_dedup(wl.dedup_objs(), stream=stream.cuda_stream)
        d2h += 4 * 5

    step()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(steps):
        step()
    torch.cuda.synchronize()
    dt = (time.perf_counter() - t) / steps
    return {"value": wl.total_records / dt, "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "ms_per_step": dt * 1e3, "steps": steps, "path": "ve_analyze_records_host (pinned; two staging buffers, H2D on a side stream overlapped with the analysis)"}


if __name__ == "__main__":
    main()
