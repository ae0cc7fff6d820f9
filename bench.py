#!/usr/bin/env python
"""bench.py — input tuples/s of a fused RA chain on 1..8 B200 (BASELINE.json metric).

Default workload (N=1): configs[1] = C2, SELECT -> PROJECT -> SELECT over 2^29
4-column int32 tuples per GPU (weak scaling: rank r owns rows [r*2^29, (r+1)*2^29)
of a 2^29*N-row relation, no data-path collective).  One step = one
rw_plan_execute of the whole fused chain over the rank's relation.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2|c1|c3|c4|c5]
    torchrun --nproc-per-node N bench.py --gpus N ...
    python bench.py --impl reference ...     # the oracle (CPU) as the reference arm

Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads  # noqa: E402

W = {"i32": 4, "u32": 4, "i64": 8, "u64": 8, "u8": 1}

CONFIGS = {
    "c1": dict(name="C1: SELECT->SELECT (50%, 50%) over 2^20 (u32 key, u32 val)", rows=workloads.C1_ROWS),
    "c2": dict(name="C2: SELECT->PROJECT->SELECT over 2^29 x 4 int32 per GPU", rows=workloads.C2_ROWS),
    "c3": dict(name="C3: JOIN (2 x 2^26, Zipf 0.5) -> SELECT -> PROJECT", rows=workloads.C3_ROWS),
    "c4": dict(name="C4: TPC-H Q1-shaped select/arith/group-by over 6e8 lineitem rows per GPU", rows=workloads.C4_ROWS),
    "cc": dict(name="Pattern (c): key SELECTs on both inputs -> JOIN (2 x 2^26, Zipf 0.5) -> SELECT -> PROJECT", rows=workloads.C3_ROWS),
    "cd": dict(name="Pattern (d) input dependence: 2 SELECTs (25% each) sharing one input of 2^29 x 4 int32 per GPU", rows=workloads.C2_ROWS),
    "cs": dict(name="Set operator (--setop, default UNION) of two sorted (u32 key, u32 val) relations, 2^26 tuples each per GPU, key-range sharded", rows=1 << 26),
    "c5": dict(name="C5: JOIN->JOIN->SELECT over three relations, 2^27 rows each per GPU (2^30 at 8 GPUs), key-range sharded", rows=1 << 27),
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="rw", choices=["rw", "reference"])
    ap.add_argument("--config", default="c2", choices=sorted(CONFIGS))
    ap.add_argument("--branches", type=int, default=2, help="cd: SELECTs sharing the input (2..4)")
    ap.add_argument("--setop", default="union", choices=["union", "intersect", "difference"])
    ap.add_argument("--rows", type=int, default=0, help="override rows per GPU (testing)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-unfused", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-rows", type=int, default=0)
    ap.add_argument("--cpu-worker", action="store_true", help=argparse.SUPPRESS)
    ap.add_argument("--cpu-start", type=int, default=0, help=argparse.SUPPRESS)
    ap.add_argument("--cpu-core", type=int, default=0, help=argparse.SUPPRESS)
    ap.add_argument("--no-sweep", action="store_true", help="skip the selectivity / size sweeps")
    ap.add_argument("--stages", type=int, default=0, help="TMA stages per CTA (0 = auto)")
    ap.add_argument("--ctas", type=int, default=0, help="CTAs per SM cap (0 = auto)")
    ap.add_argument("--defer", type=int, default=0, help="scan store delay in tiles (0 = auto)")
    ap.add_argument("--dbg", type=int, default=0, help="diagnostic ablations (not a bench value)")
    ap.add_argument("--items", type=int, default=0, help="rows per thread of the scan tile (0 = auto)")
    ap.add_argument("--variant", type=int, default=0, help="2 = 512x4, 3 = 512x8 compute threads x rows")
    ap.add_argument("--gring", type=int, default=0, help="1 = compacted-tile ring in global memory (L2)")
    ap.add_argument("--agg-mode", type=int, default=0, help="aggregate terminal switch (2 = Q1 shape through the interpreter)")
    return ap.parse_args()


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def spec_and_inputs(cfg: str, rows: int, start: int, device):
    if cfg == "c1":
        return workloads.c1_spec(), workloads.c1_inputs(rows, start, device)
    if cfg == "c2":
        return workloads.c2_spec(), workloads.c2_inputs(rows, start, device)
    if cfg == "c3":
        return workloads.c3_spec(), workloads.c3_inputs(rows, device=device)
    if cfg == "cc":
        return workloads.cc_spec(), workloads.c3_inputs(rows, device=device)
    if cfg == "c4":
        return workloads.c4_spec(), workloads.c4_inputs(rows, start, device)
    if cfg == "cd":
        return workloads.cd_spec(0.25, BRANCHES), workloads.cd_inputs(rows, start, device)
    if cfg == "cs":
        world = int(os.environ.get("WORLD_SIZE", "1"))
        return workloads.cs_spec(SETOP), workloads.cs_inputs(rows, device=device, key_space=rows * world, start=start)
    if cfg == "c5":
        world = int(os.environ.get("WORLD_SIZE", "1"))
        return workloads.c5_spec(), workloads.c5_inputs(rows, key_space=rows * world, start=start, device=device)
    raise ValueError(cfg)


BRANCHES = 2
SETOP = "union"


def spec_rows(spec, ins):
    return {k: int(v[0].numel()) for k, v in ins.items()}


class ClockSampler:
    """NVML clocks / throttle reasons sampled every 5 ms during the timed region."""

    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
               0x100: "display_clock_setting", 0x10: "sync_boost"}

    def __init__(self, index: int):
        self.samples, self.reasons, self.ok = [], set(), False
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.ok = False
        self._stop = threading.Event()

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def result(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


NOMINAL_HBM_GBS = 8000.0     # BASELINE.json "about 8 TB/s HBM3e" (DGX B200 figure; 7.7 TB/s HGX)


def measured_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            j = json.load(f)
        return float(j["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy kernel)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def ncu_traffic(cfg: str):
    """dram bytes per launch of the dominant kernel from the committed ncu capture, else None."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        with open(p) as f:
            j = json.load(f)
        return j.get(cfg)
    except Exception:
        return None


ROW_SHARDABLE = ("c1", "c2", "c4", "cd")


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_oracle_sample(cfg: str, rows: int, sample_rows: int, start: int = 0):
    """Time the oracle (single thread) on a bounded sample (rows [start, start + m)) of
    the same workload."""
    import oracle
    m = min(rows, sample_rows)
    spec, ins = spec_and_inputs(cfg, m, start, "cpu")
    rels = {}
    import numpy as np
    npt = {"i32": np.int32, "u32": np.uint32, "i64": np.int64, "u64": np.uint64, "u8": np.uint8}
    for name, inp in spec["inputs"].items():
        rels[name] = oracle.Relation(inp["types"], [c.numpy().view(npt[t]) for c, t in zip(ins[name], inp["types"])])
    t0 = time.perf_counter()
    oracle.evaluate(spec, rels)
    dt = time.perf_counter() - t0
    n_in = sum(r.n for r in rels.values())
    return n_in / dt, dt, n_in


def cpu_worker(args):
    """Child process of the CPU legs: pinned to one core, one oracle evaluation over its
    rows; prints {"n_in", "seconds"}."""
    try:
        os.sched_setaffinity(0, {args.cpu_core})
    except (AttributeError, OSError):
        pass
    os.environ["OMP_NUM_THREADS"] = "1"
    v, dt, n_in = cpu_oracle_sample(args.config, args.cpu_rows, args.cpu_rows, args.cpu_start)
    print(json.dumps({"n_in": n_in, "seconds": dt}), flush=True)
    return 0


def cpu_legs(cfg: str, rows: int, sample: int, multi: bool = True):
    """The oracle on the box's host cores: one process pinned to one core (sched_setaffinity)
    over a bounded sample, and for row-shardable chains N independent pinned processes over
    N row shards of the same size (N = the cores this process may run on).  Returns the
    cpu_baseline object."""
    import subprocess
    import oracle
    oracle.build()
    cores = sorted(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else [0]
    base = [sys.executable, os.path.abspath(__file__), "--config", cfg, "--cpu-worker"]
    if cfg == "cd":
        base += ["--branches", str(BRANCHES)]
    if cfg == "cs":
        base += ["--setop", SETOP]
    m = min(rows, sample)

    def launch(core, start):
        return subprocess.Popen(base + ["--cpu-rows", str(m), "--cpu-start", str(start), "--cpu-core", str(core)],
                                stdout=subprocess.PIPE, text=True)

    def result(pr):
        out, _ = pr.communicate()
        return json.loads([l for l in out.splitlines() if l.startswith("{")][-1])

    one = result(launch(cores[0], 0))
    v1 = one["n_in"] / one["seconds"]
    out = {"value": v1, "unit": "tuples/s", "cores": 1, "kind": "oracle", "pinned": f"core {cores[0]} (sched_setaffinity)",
           "sample": f"input tuples [0, {one['n_in']}) of the same workload, one pinned process ({one['seconds']:.2f} s)",
           "cpu_model": cpu_model()}
    if multi and cfg in ROW_SHARDABLE and len(cores) > 1 and m == sample:
        prs = [launch(c, k * m) for k, c in enumerate(cores)]
        res = [result(pr) for pr in prs]
        wall = max(r["seconds"] for r in res)
        n_all = sum(r["n_in"] for r in res)
        out["all_cores"] = {"value": n_all / wall, "unit": "tuples/s", "cores": len(cores),
                            "sample": f"{len(cores)} independent pinned processes, row shards of {m} rows each "
                                      f"(slowest {wall:.2f} s)"}
    return out


def run_reference(args):
    rank, world, local = dist_env()
    if rank != 0:
        return 0
    cfg = args.config
    rows = args.rows or CONFIGS[cfg]["rows"]
    sample = args.cpu_rows or {"c1": rows, "c2": 1 << 24, "c3": 1 << 21, "c4": 1 << 23, "c5": 1 << 21, "cd": 1 << 24, "cs": 1 << 21, "cc": 1 << 21}[cfg]
    import oracle
    oracle.build()
    try:
        os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})   # one pinned host core
    except (AttributeError, OSError):
        pass
    vals = []
    for i in range(args.warmup + args.steps):
        v, dt, n_in = cpu_oracle_sample(cfg, rows, sample)
        if i >= args.warmup:
            vals.append((v, dt, n_in))
    value = statistics.median(v for v, _, _ in vals)
    ms = statistics.median(dt for _, dt, _ in vals) * 1e3
    line = {"metric": "input tuples/sec per fused chain", "value": value, "unit": "tuples/s",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "int64" if cfg == "c4" else ("u32" if cfg in ("c1", "c3", "c5", "cs", "cc") else "i32"),
            "data": "synthetic (rwgen seeded generators)", "impl": "reference",
            "config": {"workload": CONFIGS[cfg]["name"], "sample_rows": vals[0][2],
                       "note": "reference arm = the CPU oracle (single thread) on a bounded prefix sample"},
            "cpu_baseline": {"value": value, "unit": "tuples/s", "cores": 1, "kind": "oracle",
                             "sample": f"first {vals[0][2]} input tuples of {cfg}, one pinned core",
                             "cpu_model": cpu_model()},
            "e2e": {"value": value, "unit": "tuples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def sweeps(cfg, local, stream, dev, args):
    """Selectivity sweep s in {0.1, 0.5, 0.9} for both SELECTs (Fig. 20) on C1 and C2,
    and the C1 size sweep 2^20 .. 2^30 tuples (Fig. 4): fused vs operator-at-a-time
    per point, CUDA events, L2 flushed before each step when the input fits in L2."""
    import torch
    from tests.planspec import build_gpu_plan
    dtn = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64, "u8": torch.uint8}
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    out = {}

    def point(spec, ins, steps=5):
        n = int(next(iter(ins.values()))[0].numel())
        inputs = [(n, ins[k]) for k in spec["inputs"]]
        nb = workloads.input_bytes(spec, {k: n for k in spec["inputs"]})
        res = {}
        for fuse in (True, False):
            plan, ids = build_gpu_plan(spec, device=local, stream=stream, fuse=fuse)
            node = ids[spec["out"]]
            types = plan.node_schema(node)
            outs = [torch.empty(n, dtype=dtn[t], device=dev) for t in types]
            nd = torch.zeros(1, dtype=torch.int64, device=dev)
            for _ in range(2):
                plan.execute(inputs, node, outs, n, n_dev=nd)
            ts = []
            for _ in range(steps):
                if nb < (512 << 20):
                    flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                plan.execute(inputs, node, outs, n, n_dev=nd)
                e1.record(stream)
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = statistics.median(ts)
            res["fused_ms" if fuse else "unfused_ms"] = ms
            if fuse:
                res["tuples_per_s"] = n / (ms / 1e3)
                res["out_rows"] = int(nd.item())
            del outs, plan
        res["speedup"] = res["unfused_ms"] / res["fused_ms"]
        return res

    sel = {}
    for sv in (0.1, 0.5, 0.9):
        if cfg == "c1":
            spec, ins = workloads.c1_spec(sv, sv), workloads.c1_inputs(workloads.C1_ROWS, 0, dev)
        else:
            spec, ins = workloads.c2_spec(sv, sv), workloads.c2_inputs(workloads.C2_ROWS, 0, dev)
        sel[str(sv)] = point(spec, ins)
        del ins
        torch.cuda.empty_cache()
    out["selectivity"] = sel
    if cfg == "c1":
        size = {}
        for lg in range(20, 31, 2):
            ins = workloads.c1_inputs(1 << lg, 0, dev)
            size[f"2^{lg}"] = point(workloads.c1_spec(), ins)
            del ins
            torch.cuda.empty_cache()
        out["size"] = size
    out["note"] = "median of 5 CUDA-event steps per point; speedup = operator-at-a-time / fused time"
    return out


def main():
    args = parse()
    global BRANCHES, SETOP
    BRANCHES = args.branches
    SETOP = args.setop
    if args.cpu_worker:
        return cpu_worker(args)
    if args.impl == "reference":
        return run_reference(args)
    import torch
    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    dev = f"cuda:{local}"
    pg = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device(dev))
        pg = dist
    from paper_conf_micro_wudcy12_b200 import rw
    from tests.planspec import build_gpu_plan

    cfg = args.config
    rows = args.rows or CONFIGS[cfg]["rows"]
    spec, ins = spec_and_inputs(cfg, rows, rank * rows, dev)
    nrows = spec_rows(spec, ins)
    n_in = sum(nrows.values())
    in_bytes = workloads.input_bytes(spec, nrows)
    stream = torch.cuda.current_stream()

    dtn = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64, "u8": torch.uint8}

    def make(fuse):
        plan, ids = build_gpu_plan(spec, device=local, stream=stream, fuse=fuse, stages=args.stages,
                                   ctas_per_sm=args.ctas, defer=args.defer, dbg=args.dbg, items=args.items, variant=args.variant, gring=args.gring,
                                   agg_mode=args.agg_mode)
        if "outs" in spec:
            # input-dependence fusion: one output relation per branch
            cap = max(nrows.values())
            out_types = [plan.node_schema(ids[o]) for o in spec["outs"]]
            outs = [[torch.empty(cap, dtype=dtn[t], device=dev) for t in ts] for ts in out_types]
            return plan, ids, outs, cap, out_types
        out_types = plan.node_schema(ids[spec["out"]])
        cap = {"c4": 6}.get(cfg, max(nrows.values()))
        if cfg in ("c3", "cc"):
            cap = 400_000_000 if rows == workloads.C3_ROWS else 8 * rows + 1024
        if cfg in ("c5", "cs"):
            cap = 2 * max(nrows.values()) + 4096
        outs = [torch.empty(cap, dtype=dtn[t], device=dev) for t in out_types]
        return plan, ids, outs, cap, out_types

    inputs = [(nrows[k], ins[k]) for k in spec["inputs"]]
    n_dev = torch.zeros(1, dtype=torch.int64, device=dev)
    from paper_conf_micro_wudcy12_b200 import dist as rdist

    n_devs = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in spec.get("outs", [])]

    def make_step(plan, ids, outs, cap):
        node = ids[spec["out"]]
        if "outs" in spec:
            nodes = [ids[o] for o in spec["outs"]]

            def step():
                plan.execute_multi(inputs, nodes, outs, [cap] * len(nodes), n_devs=n_devs)
                return plan.last_launches()
            return step
        if cfg == "c4" and world > 1:
            # local fused Q1, exact limb export, one NCCL all-reduce, import
            limbs = torch.empty(plan.agg_limbs(node), dtype=torch.int64, device=dev)
            loc = [torch.empty(6, dtype=o.dtype, device=dev) for o in outs]
            loc_n = torch.zeros(1, dtype=torch.int64, device=dev)

            def step():
                plan.execute(inputs, node, loc, 6, n_dev=loc_n)
                plan.agg_export(node, loc, n_dev=loc_n, limbs=limbs)
                pg.all_reduce(limbs, op=pg.ReduceOp.SUM)
                plan.agg_import(node, limbs, outs, cap, n_dev=n_dev)
                return plan.last_launches() + 2
            return step
        if cfg in ("c5", "cs") and world > 1:
            schema = {k: v["types"] for k, v in spec["inputs"].items()}
            backend = rdist.GpuBackend(local)

            def step():
                mine = rdist.exchange_all(backend, ins, schema, world)
                loc_in = [(int(mine[k][0].numel()), mine[k]) for k in spec["inputs"]]
                plan.execute(loc_in, node, outs, cap, n_dev=n_dev)
                # per relation: k_split_bounds, k_mp_pack, k_mp_samples/rank/cuts/merge
                return plan.last_launches() + 6 * len(spec["inputs"])
            return step

        def step():
            plan.execute(inputs, node, outs, cap, n_dev=n_dev)
            return plan.last_launches()
        return step

    # inputs smaller than 4x L2 (C1): flush L2 between timed steps by writing 512 MB,
    # outside each step's event pair
    flush_buf = torch.empty(512 << 20, dtype=torch.uint8, device=dev) if in_bytes < (512 << 20) else None

    def timed(step, steps, warmup):
        for _ in range(warmup):
            step()
        torch.cuda.synchronize()
        if pg:
            pg.barrier()
        torch.cuda.synchronize()
        ev0 = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
        ev1 = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
        launches = 0
        sampler = ClockSampler(local)
        with sampler:
            for i in range(steps):
                if flush_buf is not None:
                    flush_buf.zero_()
                ev0[i].record(stream)
                launches += step()
                ev1[i].record(stream)
            torch.cuda.synchronize()
        per = [ev0[i].elapsed_time(ev1[i]) for i in range(steps)]
        total_ms = sum(per)
        if pg:
            t = torch.tensor([total_ms], device=dev)
            pg.all_reduce(t, op=pg.ReduceOp.MAX)
            total_ms = float(t.item())
        return total_ms, per, launches, sampler.result()

    plan, ids, outs, cap, out_types = make(True)
    total_ms, per, launches, clocks = timed(make_step(plan, ids, outs, cap), args.steps, args.warmup)
    if "outs" in spec:
        n_outs = [int(x.item()) for x in n_devs]
        n_out = sum(n_outs)
        out_bytes = sum(nk * sum(W[t] for t in ts) for nk, ts in zip(n_outs, out_types))
    else:
        n_out = int(n_dev.item())
        out_bytes = n_out * sum(W[t] for t in out_types)
    ms_step = total_ms / args.steps
    value = n_in * world / (total_ms / 1e3 / args.steps)

    # roofline of the dominant kernel, timed as the step on the plan's stream (CUDA events).
    # C1/C2: the fused k_scan_emit is the whole step; C4: k_scan_chain<576,4,agg> (the
    # Q1 row path; k_agg_finalize is a 1-CTA epilogue of a few us); C3/C5: the join
    # kernels (k_jsplit + k_jmatch + k_jtiles + k_join_emit); algorithmic bytes = inputs
    # + output.
    alg_bytes = in_bytes + out_bytes
    peak, peak_src = measured_peak()
    kern_ms = statistics.mean(per)
    achieved = alg_bytes / (kern_ms / 1e3) / 1e9
    kname = {"c3": "k_jsplit + k_jmatch + k_jtiles + k_join_emit",
             "cc": "k_jsplit + k_jmatch (key SELECTs fused) + k_jtiles + k_join_emit",
             "c5": "exchange + 2 x (k_jsplit + k_jmatch) + k_jtiles + k_join_emit (3-input group)",
             "cs": "k_set_splits + k_set_op", "c4": "k_scan_chain<576,4,agg> (Q1 row path) + k_agg_finalize",
             "cd": "k_scan_chain<256,8,multi>"}.get(cfg, "k_scan_emit")
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "frac_nominal": achieved / NOMINAL_HBM_GBS, "nominal_peak": NOMINAL_HBM_GBS,
                "traffic": ncu_traffic(cfg), "kernel": kname,
                "alg_bytes_per_launch": alg_bytes, "peak_source": peak_src,
                "note": "achieved = (input bytes + compacted output bytes) / CUDA-event time per step; "
                        "peak = measured copy bandwidth (MEASURED_PEAKS.json hbm_gbs)"}

    par = {"c5": f"key-range shard x{world} (all_to_all)", "cs": f"key-range shard x{world} (all_to_all)",
           "c4": f"row-shard x{world} + limb all-reduce"}
    line = {"metric": "input tuples/sec per fused chain", "value": value, "unit": "tuples/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_step,
            "ms_median": statistics.median(per), "ms_min": min(per), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int64" if cfg == "c4" else ("u32" if cfg in ("c1", "c3", "c5", "cs", "cc") else "i32"),
            "data": "synthetic (rwgen seeded SplitMix64 generators, generated on device)",
            "config": {"workload": CONFIGS[cfg]["name"], "rows_per_gpu": nrows, "output_rows_per_gpu": n_out,
                       "parallelism": par.get(cfg, f"row-shard x{world}"),
                       "l2": "inputs larger than L2 (no flush needed)" if in_bytes > (1 << 28) else "L2 flushed before every step",
                       "fused": True},
            "roofline": roofline, "gpu_launches": launches, "clocks": clocks}

    if not args.no_unfused and cfg in ("c1", "c2", "c4", "c3", "cd", "cc"):
        del outs
        torch.cuda.empty_cache()
        uplan, uids, uouts, ucap, _ = make(False)
        us = max(3, args.steps // 4)
        ut, uper, ul, _ = timed(make_step(uplan, uids, uouts, ucap), us, 2)
        uv = n_in * world / (ut / 1e3 / us)
        line["unfused"] = {"value": uv, "ms_per_step": ut / us, "gpu_launches_per_step": ul / us,
                           "speedup_fused_vs_unfused": value / uv,
                           "roofline_frac_same_numerator": alg_bytes / (ut / us / 1e3) / 1e9 / peak,
                           "note": "operator at a time: every intermediate relation materialised (PROJECT copies its columns)"}
        del uouts, uplan
        torch.cuda.empty_cache()
        # stricter baseline: a PROJECT of plain column references aliases its input columns
        zplan, zids = build_gpu_plan(spec, device=local, stream=stream, fuse=False, zero_copy_project=True)
        zcap = cap
        zouts = [torch.empty(zcap, dtype=dtn[t], device=dev) for t in out_types] if "outs" not in spec else None
        if zouts is not None:
            zt, _, zl, _ = timed(make_step(zplan, zids, zouts, zcap), us, 2)
            zv = n_in * world / (zt / 1e3 / us)
            line["unfused_zero_copy"] = {"value": zv, "ms_per_step": zt / us, "gpu_launches_per_step": zl / us,
                                         "speedup_fused_vs_unfused": value / zv,
                                         "note": "operator at a time with zero-copy PROJECT (column aliases)"}
        del zouts, zplan
        torch.cuda.empty_cache()

    if not args.no_sweep and cfg in ("c1", "c2") and world == 1 and not args.rows:
        line["sweeps"] = sweeps(cfg, local, stream, dev, args)
        torch.cuda.empty_cache()

    if not args.no_e2e and cfg in ("c1", "c2", "c4"):
        # end to end through rw_plan_execute_host: pinned host inputs copied H2D and the
        # result copied D2H inside the timed region
        host_in = [(n, [c.cpu().pin_memory() for c in cols]) for n, cols in inputs]
        eplan, eids, _, ecap, etypes = None, None, None, None, None
        eplan, eids = build_gpu_plan(spec, device=local, stream=stream)
        etypes = eplan.node_schema(eids[spec["out"]])
        ecap = {"c4": 6}.get(cfg, max(nrows.values()))
        dtn = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64, "u8": torch.uint8}
        host_out = [torch.empty(ecap, dtype=dtn[t]).pin_memory() for t in etypes]
        esteps = max(2, min(args.steps, 5))
        for _ in range(1):
            eplan.execute_host(host_in, eids[spec["out"]], host_out, ecap)
        if pg:
            pg.barrier()
        t0 = time.perf_counter()
        n_e = 0
        for _ in range(esteps):
            n_e = eplan.execute_host(host_in, eids[spec["out"]], host_out, ecap)
        et = (time.perf_counter() - t0) / esteps
        if pg:
            t = torch.tensor([et], device=dev)
            pg.all_reduce(t, op=pg.ReduceOp.MAX)
            et = float(t.item())
        line["e2e"] = {"value": n_in * world / et, "unit": "tuples/s", "h2d_bytes_per_step": in_bytes,
                       "d2h_bytes_per_step": n_e * sum(W[t] for t in etypes), "ms_per_step": et * 1e3,
                       "api": "rw_plan_execute_host (pinned host buffers; 2^25-row chunks, H2D / kernel / D2H overlapped on 3 streams)"}
        del host_in, host_out

    if rank == 0 and not args.no_cpu:
        sample = args.cpu_rows or {"c1": rows, "c2": 1 << 25, "c3": 1 << 22, "c4": 1 << 23, "c5": 1 << 22, "cd": 1 << 25, "cs": 1 << 22, "cc": 1 << 22}[cfg]
        line["cpu_baseline"] = cpu_legs(cfg, rows, sample)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if pg:
        pg.barrier()
        pg.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
