"""bench.py -- value-trace analysis throughput on B200 (BASELINE.json metric).

One step = one pass of the whole hot path over the N=1
workload, BASELINE.json configs[3] -- cfg4, the largest single-GPU configuration:
LAMMPS/Castro-style f64 stencils on a 512^3 grid, 2,013,265,920 records, 48.3 GB
of trace:
  epoch 0 (hotspot3D-like): set_objects -> analyze 1.07 G records -> snapshot diff (all 6 objects) -> report
  epoch 1 (Castro slopes):  set_objects -> analyze 0.94 G records -> snapshot diff (all 6 objects) -> report
  duplicate scan over epoch 1's six objects (5 GiB of post snapshots).
Inputs are generated on the device before timing (48 GB > 126 MB L2, so no
flush is needed).  With --gpus N (torchrun) each rank analyzes its contiguous
1/N of every epoch and the ranks merge over NCCL (strong scaling).  Extra
lines (rank 0, N=1): cfg2 (configs[1]) and cfg3 (configs[2]) with their own
roofline blocks, the SURVEY 8(f) rows on cfg2's gemm epoch, and cfg5's two
halves (configs[4]).

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


# ----------------------------------------------------------------------------- workloads
# Per configuration: the epochs (one API call each), the objects whose snapshots are diffed after the
# epoch (the written ones), and the recipe's referenced pre-snapshot elements U per epoch (algorithmic
# bytes B_rec = 24 N + ew U; DESIGN.md section 7 derives each U from gen/ve_gen_core.h).
CONFIGS = {
    "cfg4": {"code": ("CFG4", 0), "seed": 4, "epochs": (0, 1), "diff": {0: [1], 1: [3]}, "hcap": 1 << 22,
             "workload": "cfg4: LAMMPS/Castro-style f64 stencils on a 512^3 grid (hotspot3D-like 7-point + "
                         "Castro slopes-like), BASELINE configs[3]",
             # e0: T_in and T_out referenced in full; e1: a, vol, s in full and xc (512 elements)
             "U": lambda: [2 * 512 ** 3, 3 * 512 ** 3 + 512], "ew": 8},
    "cfg2": {"code": ("CFG2", None), "seed": 2, "epochs": (0, 1), "diff": {0: [2], 1: [2]}, "hcap": 1 << 22,
             "workload": "cfg2: Darknet YOLOv4 conv layer trace (fill_ongpu + gemm beta=1; M=256 K=1152 "
                         "N=5776 batch 4), BASELINE configs[1]",
             "U": lambda: [5914624, 294912 + 6653952 + 5914624], "ew": 4},
}
HEADLINE = "cfg4"


def cfg_code(name):
    from gen import vegen as G
    c, shift = CONFIGS[name]["code"]
    base = getattr(G, c)
    return base if shift is None else G.scaled(base, shift)


class Workload:
    """One configuration on the device: this rank's records of each epoch + the epoch's snapshots."""

    def __init__(self, name, rank, world, device):
        import torch
        from gen import vegen as G
        self.name, self.G, self.torch = name, G, torch
        spec = CONFIGS[name]
        self.spec = spec
        cfg = cfg_code(name)
        self.cfg, self.seed = cfg, spec["seed"]
        self.device = device
        self.epochs = []
        stream = torch.cuda.current_stream().cuda_stream
        self.total_records = 0
        for ep in spec["epochs"]:
            inf = G.info(cfg, ep)
            n = inf["n_records"]
            self.total_records += n
            lo, hi = n * rank // world, n * (rank + 1) // world   # = ve.rank_chunk
            recs = torch.empty((hi - lo) * REC_BYTES, dtype=torch.uint8, device=device)
            G.records_device(cfg, ep, self.seed, lo, hi - lo, recs.data_ptr(), stream)
            objs = []
            for i, o in enumerate(G.objects(cfg, ep)):
                pre = torch.empty(o["size"], dtype=torch.uint8, device=device)
                post = torch.empty(o["size"], dtype=torch.uint8, device=device)
                G.snapshot_device(cfg, ep, self.seed, i, 0, pre.data_ptr(), stream)
                G.snapshot_device(cfg, ep, self.seed, i, 1, post.data_ptr(), stream)
                objs.append({"base": o["base"], "size": o["size"], "id": o["id"], "elem_width": o["elem_width"],
                             "pre": pre, "post": post})
            self.epochs.append({"epoch": ep, "n_pcs": inf["n_pcs"], "lo": lo, "n": hi - lo, "recs": recs,
                                "objs": objs, "n_total": n, "diff": spec["diff"][ep]})
        torch.cuda.synchronize()
        self.n_pcs = max(e["n_pcs"] for e in self.epochs)
        self.max_objects = max(len(e["objs"]) for e in self.epochs) + 1
        self.trace_bytes = self.total_records * REC_BYTES
        U = spec["U"]()
        self.alg_bytes_epoch = [e["n_total"] * REC_BYTES + spec["ew"] * u for e, u in zip(self.epochs, U)]

    def dedup_objs(self):
        """S11 over the last epoch's post snapshots (cfg2: + the zero x_gpu twin of output, P3)."""
        o = self.epochs[-1]["objs"]
        out = [{"base": x["base"], "size": x["size"], "id": x["id"], "elem_width": x["elem_width"], "pre": None,
                "post": x["post"]} for x in o]
        if self.name == "cfg2":
            out.append({"base": 0x7f9000000000, "size": o[2]["size"], "id": len(o), "elem_width": 4, "pre": None,
                        "post": self.epochs[0]["objs"][2]["post"]})
        return out

    def spot_check(self, reps, groups):
        """parity at full size: the recipe's closed forms (tests/cfg34.py for cfg4, cfg2's below)"""
        if self.name == "cfg4":
            from tests import cfg34
            ok = True
            for e, rep in zip(self.epochs, reps):
                k = {f: rep.keys[f] for f in rep.keys.dtype.names}
                k["top_bits"], k["top_count"] = rep.topk["bits"], rep.topk["count"]
                ok = ok and not cfg34.check_cfg4(k, int(rep.globals["n_records"]), 0, e["epoch"], rep.objects)
            return {"cfg4_closed_forms": bool(ok), "dedup_all_distinct": len(set(int(g) for g in groups)) == len(groups)}
        k0, k1 = reps[0].keys, reps[1].keys
        return {"fill_redundant_stores": int(k0["n_st_eq_pre"][0]) == self.epochs[0]["n_total"],
                "c_load_single_zero": bool(k1["single_zero"][3]) and int(k1["n_ld_eq_pre"][3]) == 5914624,
                "a_loads": int(k1["n_ld"][1]) == 107347968, "b_loads": int(k1["n_ld"][2]) == 106463232,
                "dedup_output_xgpu": int(groups[4]) == 3 and int(groups[3]) == 3}


def run_step(ctx, wl, tstream, ev_pairs=None, comm=None):
    """One pass of the hot path over every epoch (S1-S13): set_objects, analyze, (rank merge), snapshot
    diff of every object (sharded by object over the ranks), report; then the duplicate-object scan
    (sharded by object)."""
    stream = tstream.cuda_stream
    reps = []
    for i, e in enumerate(wl.epochs):
        ctx.set_objects(e["objs"])
        if ev_pairs is not None:
            ev_pairs[i][0].record(tstream)
        ctx.analyze_records(e["recs"], e["n"], stream=stream)
        if ev_pairs is not None:
            ev_pairs[i][1].record(tstream)
        if comm is not None:
            ctx.merge(comm=comm, stream=stream)
        # S10 of every object with both snapshots, sharded by object over the ranks (N = 1: all local)
        ctx.snapshot_diff_all(comm=comm, stream=stream)
        reps.append(ctx.report())
    groups = ctx.object_dedup(wl.dedup_objs(), comm=comm, stream=stream)   # S11, sharded by object
    return reps, groups


# ----------------------------------------------------------------------------- CPU oracle arm
ORACLE_SAMPLE = "cfg4 recipe at 1/4 scale per axis (128^3 grid, epoch 0: 16,777,216 records, 16 MiB objects)"


def oracle_sample():
    """Bounded sample of the headline workload for the oracle: the cfg4 recipe at shift 2 (128^3 grid;
    the same kernels, PCs, objects and value rules), epoch 0, all records, full snapshots."""
    from gen import vegen as G
    from oracle import oracle as O
    cfg = G.scaled(G.CFG4, 2)
    inf = G.info(cfg, 0)
    recs = G.records_host(cfg, 0, 4, 0, inf["n_records"])
    objs = []
    for i, o in enumerate(G.objects(cfg, 0)):
        d = dict(o)
        d["pre"] = G.snapshot_host(cfg, 0, 4, i, 0)
        d["post"] = G.snapshot_host(cfg, 0, 4, i, 1)
        objs.append(d)
    return O, O.make_config(inf["n_pcs"]), objs, recs


def time_oracle():
    O, cfg, objs, recs = oracle_sample()
    t = time.perf_counter()
    O.analyze(cfg, objs, recs)
    dt = time.perf_counter() - t
    return len(recs) / dt, dt, len(recs)


def cpu_info():
    model = "unknown"
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"model": model, "nproc": os.cpu_count(), "threads_used": 1,
            "pinning": "none (single-threaded oracle; the process is not taskset)"}


def reference_arm(args, rank, world):
    """--impl reference: the CPU oracle, as it stands, on the host (rank 0 only)."""
    if rank != 0:
        return
    O, cfg, objs, recs = oracle_sample()
    n_sample = len(recs)
    for _ in range(args.warmup):
        O.analyze(cfg, objs, recs[: max(1, n_sample // 64)])
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
            "config": workload_config(HEADLINE, sample=n_sample),
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": ORACLE_SAMPLE,
                             "cpu": cpu_info()},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def workload_config(name, sample=None, world=1):
    from gen import vegen as G
    spec = CONFIGS[name]
    cfg = cfg_code(name)
    n = sum(G.info(cfg, ep)["n_records"] for ep in spec["epochs"])
    c = {"workload": spec["workload"], "records": n, "trace_bytes": n * REC_BYTES,
         "epochs": len(spec["epochs"]),
         "l2": "inputs larger than L2 (%.1f GB trace vs 126 MB), no flush" % (n * REC_BYTES / 1e9),
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


def measure_config(ve, name, rank, world, dev, steps, warmup, comm=None, clocks=False):
    """Time `steps` steps of configuration `name` (CUDA events on the launch stream, after `warmup`)."""
    import torch
    wl = Workload(name, rank, world, dev)
    ctx = ve.Context(n_pcs=wl.n_pcs, max_objects=wl.max_objects,
                     hist_capacity=int(os.environ.get("VE_BENCH_HCAP", CONFIGS[name]["hcap"])), device=dev.index or 0)
    stream = torch.cuda.current_stream()
    for _ in range(warmup):
        run_step(ctx, wl, stream, comm=comm)
    torch.cuda.synchronize()
    ne = len(wl.epochs)
    evs = [[[torch.cuda.Event(enable_timing=True) for _ in range(2)] for _ in range(ne)] for _ in range(steps)]
    clk = Clocks(dev.index or 0) if clocks else None
    launches0 = ve.kernel_launches()
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    if clk:
        clk.start()
        time.sleep(0.3)
    start.record(stream)
    for k in range(steps):
        reps, groups = run_step(ctx, wl, stream, ev_pairs=evs[k], comm=comm)
    end.record(stream)
    torch.cuda.synchronize()
    cl = clk.stop() if clk else None
    launches = ve.kernel_launches() - launches0
    ms = start.elapsed_time(end)
    if world > 1:
        ms = max_over_ranks(ms, device=dev)
    ms_step = ms / steps
    an_ms = [statistics.mean(evs[k][i][0].elapsed_time(evs[k][i][1]) for k in range(steps)) for i in range(ne)]
    res = {"wl": wl, "ctx": ctx, "ms_step": ms_step, "value": wl.total_records / (ms_step / 1e3),
           "an_ms": an_ms, "launches": launches, "clocks": cl, "spot": wl.spot_check(reps, groups)}
    return res


def roofline_block(res, world, peak, peak_src, traffic):
    """Dominant kernel: k_analyze over every epoch of the step (CUDA events around ve_analyze_records:
    K1 plus its drain and line-fold launches).  achieved = algorithmic bytes of the epochs (24 N + ew U)
    / their summed analyze time."""
    wl = res["wl"]
    alg = sum(wl.alg_bytes_epoch) / world
    t = sum(res["an_ms"]) / 1e3
    achieved = alg / t / 1e9
    return {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
            "traffic": traffic,
            "traffic_source": ("ncu --set full capture of this command's timed step (scripts/r2_final.sh), "
                               "profiles/r02_k_analyze_traffic.json; per launch, bytes moved" if traffic else None),
            "kernel": "k_analyze2 / k_analyze (every epoch's ve_analyze_records)",
            "peak_source": peak_src, "ms_per_launch": [round(x, 4) for x in res["an_ms"]],
            "alg_bytes_per_launch": [b / world for b in wl.alg_bytes_epoch],
            "alg_bytes_rule": "24 B per record + element width x U (distinct pre-snapshot elements referenced)"}


def traffic_of(name):
    """dram__bytes_read.sum + dram__bytes_write.sum per analyze launch (the step's epochs), from the committed
    ncu --set full capture of the same command (profiles/r02_k_analyze_traffic.json, scripts/r2_final.sh):
    a list per epoch, or None when no capture exists for the configuration."""
    prof = os.path.join(ROOT, "profiles", "r02_k_analyze_traffic.json")
    try:
        return json.load(open(prof)).get(name)
    except Exception:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-f1", action="store_true")
    ap.add_argument("--no-cfg5", action="store_true")
    ap.add_argument("--cfg5-mode", default="units", choices=["units", "contexts"],
                    help="cfg5 records: batched units per launch (default) or one context per kernel x 8 threads")
    ap.add_argument("--no-extra", action="store_true", help="skip the cfg2 / cfg3 lines")
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
    comm = ve.nccl_comm_from_torch(rank, world) if world > 1 else None
    peak, peak_src = hbm_peak()

    res = measure_config(ve, HEADLINE, rank, world, dev, args.steps, args.warmup, comm=comm, clocks=True)
    wl = res["wl"]
    roof = roofline_block(res, world, peak, peak_src, traffic_of(HEADLINE))
    single = rank == 0 and world == 1

    e2e = None
    if not args.no_e2e and single:
        e2e = measure_e2e(ve, res["ctx"], wl, max(1, min(args.steps, 2)))
    res["ctx"].close()
    del res["ctx"], res["wl"], wl
    torch.cuda.empty_cache()

    extra = {}
    if single and not args.no_extra:
        r2 = measure_config(ve, "cfg2", 0, 1, dev, max(3, args.steps), 2)
        extra["cfg2"] = {"workload": CONFIGS["cfg2"]["workload"], "records": r2["wl"].total_records,
                         "ms_per_step": r2["ms_step"], "records_per_s": r2["value"],
                         "trace_gbs": r2["value"] * REC_BYTES / 1e9,
                         "roofline": roofline_block(r2, 1, peak, peak_src, traffic_of("cfg2")),
                         "parity_spot_check": r2["spot"]}
        f1 = None if args.no_f1 else measure_next_rows(ve, r2["ctx"], r2["wl"], torch.cuda.current_stream(), peak)
        r2["ctx"].close()
        del r2
        torch.cuda.empty_cache()
        extra["cfg3"] = measure_cfg3(ve, torch.cuda.current_stream(), peak)
        extra["next_rows"] = f1
        extra["f4_value_flow_graph"] = measure_vfg(ve)
    dd5 = r5 = None
    if single and not args.no_cfg5:
        dd5 = measure_cfg5_dedup(ve, torch.cuda.current_stream(), peak)
    if not args.no_cfg5:          # every rank: its LPT share of the 4000 kernels (weak-style partition)
        if args.cfg5_mode == "units":
            r5 = measure_cfg5_units(ve, torch.cuda.current_stream(), peak, rank, world, dev)
        else:
            r5 = measure_cfg5_records(ve, torch.cuda.current_stream(), peak, rank, world, dev)

    cpu = None
    if not args.no_cpu and single:
        rate, dt, ns = time_oracle()
        cpu = {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": ORACLE_SAMPLE + f"; {dt:.1f} s single-threaded", "cpu": cpu_info()}

    if rank == 0:
        line = {"metric": METRIC, "value": res["value"], "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": res["ms_step"], "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": "u64",
                "data": "synthetic (seeded counter-based generator, cfg4 recipe; inputs generated on the device)",
                "config": workload_config(HEADLINE, world=world),
                "trace_gbs": res["value"] * REC_BYTES / 1e9,
                "roofline": roof,
                "analyze_ms_per_step": [round(x, 4) for x in res["an_ms"]],
                "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": res["launches"], "clocks": res["clocks"],
                "parity_spot_check": res["spot"], "extra_configs": extra, "cfg5_dedup": dd5, "cfg5_records": r5}
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


def measure_cfg3(ve, stream, peak):
    """BASELINE configs[2] (cfg3, PyTorch op mix: 4 iterations x 264 M records), full size, outside the
    step: per iteration the records and snapshots are generated on the device (untimed), then
    set_objects + ve_analyze_records + ve_report are timed with CUDA events (second pass on a warm
    context), with events around ve_analyze_records for the roofline (trace bytes only: U, at most the
    0.9 GB of snapshots, is not counted).  Parity at full size: the recipe's closed forms (tests/cfg34.py)."""
    import torch
    from gen import vegen as G
    from tests import cfg34
    sp = stream.cuda_stream
    cfg = G.scaled(G.CFG3, 0)
    tot_n, tot_ms, an_ms, ok = 0, 0.0, 0.0, True
    for seed in (3, 4, 5, 6):
        inf = G.info(cfg, 0)
        n = inf["n_records"]
        dobjs = []
        for i, o in enumerate(G.objects(cfg, 0)):
            d = {k: o[k] for k in ("base", "size", "id", "elem_width")}
            for side in ("pre", "post"):
                t = torch.empty(o["size"], dtype=torch.uint8, device="cuda")
                G.snapshot_device(cfg, 0, seed, i, side == "post", t.data_ptr(), sp)
                d[side] = t
            dobjs.append(d)
        recs = torch.empty(n * REC_BYTES, dtype=torch.uint8, device="cuda")
        G.records_device(cfg, 0, seed, 0, n, recs.data_ptr(), sp)
        ctx = ve.Context(n_pcs=inf["n_pcs"], max_objects=len(dobjs), hist_capacity=1 << 25)
        for _ in range(2):               # pass 0 warms the context (allocations, pools), pass 1 is timed
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            x, y = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            ctx.set_objects(dobjs)
            x.record(stream)
            ctx.analyze_records(recs, n, stream=sp)
            y.record(stream)
            rep = ctx.report()
            b.record(stream)
            torch.cuda.synchronize()
        tot_ms += a.elapsed_time(b)
        an_ms += x.elapsed_time(y)
        tot_n += n
        if seed == 3:
            k = {f: rep.keys[f] for f in rep.keys.dtype.names}
            k["top_bits"], k["top_count"] = rep.topk["bits"], rep.topk["count"]
            ok = ok and not cfg34.check_cfg3(k, int(rep.globals["n_records"]), 0, rep.objects)
        ctx.close()
        del dobjs, recs
        torch.cuda.empty_cache()
    gbs = tot_n * REC_BYTES / (tot_ms / 1e3) / 1e9
    ach = tot_n * REC_BYTES / (an_ms / 1e3) / 1e9
    return {"workload": "cfg3: PyTorch op mix (embedding, elementwise, reductions, index_select, zeros_like + "
                        "zero_), 4 iterations, BASELINE configs[2]",
            "records": tot_n, "ms": tot_ms, "records_per_s": tot_n / (tot_ms / 1e3), "trace_gbs": gbs,
            "trace_frac_of_hbm_peak": gbs / peak, "closed_forms_ok": ok,
            "roofline": {"bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                         "traffic": None, "kernel": "k_analyze2 (4 launches)", "ms_per_launch": an_ms / 4,
                         "alg_bytes_rule": "24 B per record (U not counted)"},
            "timed": "set_objects + analyze + report per iteration (no diff / dedup), second pass on a warm context"}


def measure_vfg(ve):
    """SURVEY 8(f) f4 on BASELINE configs[4]'s API-event log (tests/workloads.cfg5_api_log: 1000 objects,
    4000 launches from 64 call paths): host-side graph build (Def 5.1) and important graph (Def 5.3,
    edges >= 16 MiB, vertices invoked >= 70 times) -- libve's host code, wall time."""
    from tests import workloads as W
    lg = W.cfg5_api_log()
    t = time.perf_counter()
    g = ve.ValueFlowGraph.build(lg)
    tb = time.perf_counter() - t
    t = time.perf_counter()
    gi = g.important(16 << 20, 70)
    ti = time.perf_counter() - t
    return {"events": len(lg), "vertices": len(g.vertices), "edges": len(g.edges),
            "important_vertices": len(gi.vertices), "important_edges": len(gi.edges),
            "build_ms": 1e3 * tb, "important_ms": 1e3 * ti, "where": "host (libve C++), not a GPU kernel"}


def measure_cfg5_dedup(ve, stream, peak, reps=3):
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
    ctx = ve.Context(n_pcs=1, max_objects=1)
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
    ctx.close()
    del dobjs
    torch.cuda.empty_cache()
    return {"workload": "cfg5 duplicate-object scan: 1000 objects, 50 log-uniform size classes over [64 KiB, 512 MiB] "
                        "rescaled to 20 GiB, 30% zero / 10% copies / 5% one-bit flips / 55% random",
            "objects": len(objs), "bytes": total, "ms": ms,
            "alg_bytes": alg, "alg_gbs": alg / (ms / 1e3) / 1e9, "frac_of_hbm_peak": alg / (ms / 1e3) / 1e9 / peak,
            "groups": len(set(want)), "parity_closed_form": [int(x) for x in g] == want}


def measure_cfg5_records(ve, stream, peak, rank=0, world=1, dev=None, workers=8, min_wpw=32):
    """BASELINE configs[4] (cfg5), records half: 4000 independent kernels, 10^9 records in total (4..64 PCs,
    1..4 objects, 2,987 .. 1,676,166 records each; gen/ve_gen_core.h veg_cfg5_record).  All records and
    snapshots are generated on the device first (untimed, 24 GB + 2 x 4 GB); the timed region is the
    per-kernel analysis a user runs -- ve_set_objects + ve_analyze_records + ve_report for every kernel.
    The kernels are independent units, so `workers` contexts run side by side, each in its own host
    thread on its own CUDA stream (no device-wide synchronisation in libve: a ctx waits only for its own
    work), taking kernels longest-first from a shared queue; their analysis launches use only the CTAs
    that give each warp >= 32 windows (ve_config.min_windows_per_warp), so several run at once.  The
    timed region is bracketed by CUDA events (a start event every worker stream waits on, an end event
    after every worker stream's last work); events around each ve_analyze_records give the analysis
    share.  Parity at full size: the recipe's closed forms (tests/cfg5k.py) on every 50th kernel
    (kernel-by-kernel oracle parity is tests/test_gpu_cfg5.py)."""
    import threading
    import torch
    from gen import vegen as G
    from tests import cfg5k
    sp = stream.cuda_stream
    cfg, seed, K = G.scaled(G.CFG5, 0), 5, 4000
    infos = [G.info(cfg, k) for k in range(K)]
    n_all = sum(i["n_records"] for i in infos)
    # N > 1: the kernels are independent units -- each rank takes its longest-processing-time-first
    # share by record count (ve.lpt_assign: the same plan on every rank, no data-path collective)
    owner = ve.lpt_assign([i["n_records"] for i in infos], world)
    mine = [k for k in range(K) if owner[k] == rank]
    n_tot = sum(infos[k]["n_records"] for k in mine)
    recs = torch.empty(n_tot * REC_BYTES, dtype=torch.uint8, device="cuda")
    objs_of = {k: G.objects(cfg, k) for k in mine}
    snap_tot = sum(o["size"] for objs in objs_of.values() for o in objs)
    snaps = torch.empty(2 * snap_tot, dtype=torch.uint8, device="cuda")
    r0, s0, plan = 0, 0, []
    for k in mine:
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
        plan.append((k, recs[r0 * REC_BYTES:(r0 + n) * REC_BYTES], n, dobjs))
        r0 += n
    order = sorted(range(len(plan)), key=lambda j: -plan[j][2])      # longest first
    W = max(1, min(workers, len(plan)))
    streams = [torch.cuda.Stream() for _ in range(W)]
    mw = min_wpw if W > 1 else 0
    ctxs = [ve.Context(n_pcs=64, max_objects=4, hist_capacity=1 << 22, min_windows_per_warp=mw) for _ in range(W)]
    for w in range(W):                                             # warm every context (untimed)
        _, buf, n, dobjs = plan[order[-1 - w]]
        ctxs[w].set_objects(dobjs)
        ctxs[w].analyze_records(buf, n, stream=streams[w].cuda_stream)
        ctxs[w].report().close()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in plan]
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ends = [torch.cuda.Event() for _ in range(W)]
    got, errors = {}, []
    nxt = [0]
    lock = threading.Lock()

    def work(w):
        ctx, st = ctxs[w], streams[w]
        try:
            st.wait_event(a)
            while True:
                with lock:
                    if nxt[0] >= len(order):
                        break
                    j = order[nxt[0]]
                    nxt[0] += 1
                k, buf, n, dobjs = plan[j]
                ctx.set_objects(dobjs)
                ev[j][0].record(st)
                ctx.analyze_records(buf, n, stream=st.cuda_stream)
                ev[j][1].record(st)
                rep = ctx.report()
                if k % 50 == 0:
                    got[k] = ({f: rep.keys[f].copy() for f in ("n_ld", "n_st", "n_ld_eq_pre", "n_st_eq_pre", "raw_min",
                                                               "raw_max", "single_zero", "single_value")},
                              int(rep.globals["n_records"]))
                rep.close()
            ends[w].record(st)
        except Exception as e:      # noqa: BLE001  (reported below)
            errors.append(repr(e))
            ends[w].record(st)

    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    a.record(stream)
    th = [threading.Thread(target=work, args=(w,)) for w in range(W)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    for e in ends:
        stream.wait_event(e)
    b.record(stream)
    torch.cuda.synchronize()
    if errors:
        raise RuntimeError("cfg5 records worker failed: " + errors[0])
    ms = a.elapsed_time(b)
    an_ms = sum(x.elapsed_time(y) for x, y in ev)
    if world > 1:
        ms = max_over_ranks(ms, device=dev)
    bad, checked = [], 0
    for k, (keys, nrec) in got.items():
        bad += cfg5k.check_cfg5_kernel(keys, nrec, cfg, k)
        checked += 1
    for c in ctxs:
        c.close()
    del plan, recs, snaps
    torch.cuda.empty_cache()
    gbs = n_all * REC_BYTES / (ms / 1e3) / 1e9
    return {"workload": "cfg5 records: 4000 kernels, 4-64 PCs with cfg1 roles, 1-4 objects, 10^9 records",
            "kernels": K, "records": n_all, "ranks": world, "partition": "longest-processing-time-first by records "
            "(ve.lpt_assign), independent kernels, no data-path collective", "this_rank_kernels": len(mine),
            "snapshot_bytes_this_rank": 2 * snap_tot, "ms": ms, "workers": W, "min_windows_per_warp": mw,
            "records_per_s": n_all / (ms / 1e3), "trace_gbs": gbs, "trace_frac_of_hbm_peak": gbs / peak / world,
            "analyze_ms_this_rank_sum_over_workers": an_ms, "closed_forms_kernels_checked": checked,
            "closed_forms_ok": not bad, "closed_form_mismatches": bad[:5],
            "timed": f"set_objects + analyze + report per kernel, {W} contexts in {W} host threads on {W} streams "
                     "(longest kernel first from a shared queue), CUDA events around the whole, max over ranks"}


def measure_cfg5_units(ve, stream, peak, rank=0, world=1, dev=None, batch=250, workers=2):
    """BASELINE configs[4] (cfg5), records half, batched: the same 4000 independent kernels (10^9 records)
    analysed `batch` kernels per launch through ve_set_units + ve_analyze_units + one ve_report per batch
    (each kernel a unit: its own PC keys and objects, exactly as if analysed alone -- tests/test_gpu_units.py),
    `workers` contexts in host threads on their own streams taking batches from a shared queue.  Records
    and snapshots are generated on the device first (untimed; every kernel's records 16-byte aligned);
    the timed region is bracketed by CUDA events (start event waited on by every worker stream, end event
    after each worker's last work), max over ranks.  Closed forms (tests/cfg5k.py) on every 50th kernel,
    from its key slice of the batch report."""
    import threading
    import torch
    from gen import vegen as G
    from tests import cfg5k
    sp = stream.cuda_stream
    cfg, seed, K = G.scaled(G.CFG5, 0), 5, 4000
    infos = [G.info(cfg, k) for k in range(K)]
    n_all = sum(i["n_records"] for i in infos)
    owner = ve.lpt_assign([i["n_records"] for i in infos], world)
    mine = [k for k in range(K) if owner[k] == rank]
    roff, tot = {}, 0
    for k in mine:                                  # 16-byte aligned records: even record offsets
        roff[k] = tot
        tot += infos[k]["n_records"] + (infos[k]["n_records"] & 1)
    recs = torch.empty(max(tot, 2) * REC_BYTES, dtype=torch.uint8, device="cuda")
    objs_of = {k: G.objects(cfg, k) for k in mine}
    snap_tot = sum(o["size"] for objs in objs_of.values() for o in objs)
    snaps = torch.empty(2 * snap_tot, dtype=torch.uint8, device="cuda")
    s0, plan = 0, {}
    for k in mine:
        n = infos[k]["n_records"]
        G.records_device(cfg, k, seed, 0, n, recs.data_ptr() + roff[k] * REC_BYTES, sp)
        dobjs = []
        for i, o in enumerate(objs_of[k]):
            d = {f: o[f] for f in ("base", "size", "id", "elem_width")}
            for side in ("pre", "post"):
                t = snaps[s0:s0 + o["size"]]
                s0 += o["size"]
                G.snapshot_device(cfg, k, seed, i, side == "post", t.data_ptr(), sp)
                d[side] = t
            dobjs.append(d)
        plan[k] = (recs.data_ptr() + roff[k] * REC_BYTES, n, infos[k]["n_pcs"], dobjs)
    batches = [mine[i:i + batch] for i in range(0, len(mine), batch)]
    prep = []
    for b in batches:                               # per batch: the units' objects (ids shifted) and PC bases
        uobjs, units, pcb, ob, slices = [], [], 0, 0, {}
        for k in b:
            ptr, n, npc, dobjs = plan[k]
            uobjs.append([dict(d, id=d["id"] + ob) for d in dobjs])
            units.append((ptr, n, pcb, npc))
            slices[k] = (pcb, npc, n)
            pcb += npc
            ob += len(dobjs)
        prep.append((uobjs, units, pcb, ob, slices))
    W = max(1, min(workers, len(prep)))
    max_pcs = max(p[2] for p in prep)
    max_obj = max(p[3] for p in prep)
    streams = [torch.cuda.Stream() for _ in range(W)]
    ctxs = [ve.Context(n_pcs=max_pcs, max_objects=max_obj, hist_capacity=1 << 25) for _ in range(W)]
    for w in range(W):                              # warm every context on the last batch (untimed)
        uobjs, units, _, _, _ = prep[-1]
        ctxs[w].set_units(uobjs)
        ctxs[w].analyze_units(units, stream=streams[w].cuda_stream)
        ctxs[w].report().close()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ends = [torch.cuda.Event() for _ in range(W)]
    got, errors, nxt, lock = {}, [], [0], threading.Lock()
    nrec_seen = [0]

    def work(w):
        ctx, st = ctxs[w], streams[w]
        try:
            st.wait_event(a)
            while True:
                with lock:
                    if nxt[0] >= len(prep):
                        break
                    j = nxt[0]
                    nxt[0] += 1
                uobjs, units, _, _, slices = prep[j]
                ctx.set_units(uobjs)
                ctx.analyze_units(units, stream=st.cuda_stream)
                rep = ctx.report()
                with lock:
                    nrec_seen[0] += int(rep.globals["n_records"])
                for k, (pcb, npc, n) in slices.items():
                    if k % 50 == 0:
                        got[k] = ({f: rep.keys[f][pcb:pcb + npc].copy() for f in
                                   ("n_ld", "n_st", "n_ld_eq_pre", "n_st_eq_pre", "raw_min", "raw_max", "single_zero",
                                    "single_value")}, n)
                rep.close()
            ends[w].record(st)
        except Exception as e:      # noqa: BLE001  (reported below)
            errors.append(repr(e))
            ends[w].record(st)

    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    a.record(stream)
    th = [threading.Thread(target=work, args=(w,)) for w in range(W)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    for e in ends:
        stream.wait_event(e)
    b.record(stream)
    torch.cuda.synchronize()
    if errors:
        raise RuntimeError("cfg5 units worker failed: " + errors[0])
    ms = a.elapsed_time(b)
    if world > 1:
        ms = max_over_ranks(ms, device=dev)
    bad, checked = [], 0
    for k, (keys, nrec) in got.items():
        bad += cfg5k.check_cfg5_kernel(keys, nrec, cfg, k)
        checked += 1
    n_mine = sum(infos[k]["n_records"] for k in mine)
    if nrec_seen[0] != n_mine:
        bad.append(f"batch reports counted {nrec_seen[0]} records, expected {n_mine}")
    for c in ctxs:
        c.close()
    n_batches = len(prep)
    del plan, recs, snaps, prep
    torch.cuda.empty_cache()
    gbs = n_all * REC_BYTES / (ms / 1e3) / 1e9
    return {"workload": "cfg5 records: 4000 kernels, 4-64 PCs with cfg1 roles, 1-4 objects, 10^9 records",
            "kernels": K, "records": n_all, "ranks": world, "this_rank_kernels": len(mine),
            "partition": "longest-processing-time-first by records (ve.lpt_assign), independent kernels",
            "mode": f"units: {batch} kernels per ve_analyze_units launch and per report, {W} contexts in host "
                    "threads on their own streams", "batches": n_batches, "ms": ms,
            "records_per_s": n_all / (ms / 1e3), "trace_gbs": gbs, "trace_frac_of_hbm_peak": gbs / peak / world,
            "closed_forms_kernels_checked": checked, "closed_forms_ok": not bad, "closed_form_mismatches": bad[:5],
            "timed": "set_units + analyze_units + report per batch, CUDA events around the whole, max over ranks"}


def measure_e2e(ve, ctx, wl, steps):
    """Same metric through the public API from pinned HOST buffers: every step copies each epoch's records
    (ve_analyze_records_host: two device staging buffers, H2D on a side stream overlapped with the
    analysis) and its pre / post snapshots H2D, and reads the reports and dedup groups back (D2H)."""
    import torch
    host = []
    h2d = 0
    try:
        for e in wl.epochs:
            hr = torch.empty(e["recs"].numel(), dtype=torch.uint8, pin_memory=True)
            hr.copy_(e["recs"])
            snaps = [(torch.empty(o["size"], dtype=torch.uint8, pin_memory=True).copy_(o["pre"]),
                      torch.empty(o["size"], dtype=torch.uint8, pin_memory=True).copy_(o["post"])) for o in e["objs"]]
            host.append((hr, snaps))
            h2d += hr.numel() + sum(2 * o["size"] for o in e["objs"])
    except RuntimeError as ex:                    # host memory: report why instead of failing the bench
        del host
        return {"value": None, "unit": UNIT, "error": f"pinned host buffers: {ex}"[:200]}
    torch.cuda.synchronize()
    d2h = 0
    stream = torch.cuda.current_stream()

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
            d2h += ctx.snapshot_diff_all(stream=stream.cuda_stream).nbytes
            rep = ctx.report()
            d2h += rep.keys.nbytes + rep.topk.nbytes + rep.objects.nbytes + 32
        g = ctx.object_dedup(wl.dedup_objs(), stream=stream.cuda_stream)
        d2h += 4 * len(g)

    step()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(steps):
        step()
    torch.cuda.synchronize()
    dt = (time.perf_counter() - t) / steps
    return {"value": wl.total_records / dt, "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
            "ms_per_step": dt * 1e3, "steps": steps,
            "path": "ve_analyze_records_host (pinned; two staging buffers, H2D on a side stream overlapped with "
                    "the analysis) + snapshot H2D + report / dedup D2H"}


if __name__ == "__main__":
    main()
