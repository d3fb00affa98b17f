#!/usr/bin/env python
"""Benchmark of the nested-method correlated-subquery hot path on B200.

Metric (BASELINE.json): outer tuples/s (+ query latency, roofline fraction).

Headline workload (default): BASELINE.json configs[4], "C5" -- the
non-equality Query 1 (``R.col1 > S.col1``, which cannot be
unnested) with MIN, at |R| = |S| = 16M int32: 2.56e14 (r, s) pairs
on the tiled nested-loop kernel.  It is the largest single-GPU config (the
others are parity cases or side keys).  One step is one pass of the whole hot
path over that batch:

  outer scan (R') -> inner scan (S') -> tiled nested loop (the subquery for
  every outer tuple) -> aggregate finalize + outer comparison -> compaction
  of the survivors [-> at N > 1: gather of the survivors to rank 0].

N GPUs (strong scaling, §8(e)): ONE R is sharded in contiguous row blocks,
S is broadcast once (NCCL) into every rank's arena (resident input), each
rank runs the step on its shard, and the survivors are gathered to rank 0
every step.  After the timed region rank 0 checks that the gathered
survivors are identical to the whole-R result of the 1-GPU index path (a
different kernel: sorted index + prefix aggregates), i.e. that the N-GPU
result equals the 1-GPU result (T7).

value       = |R| outer tuples per plan x plans / step time (max over ranks),
              inputs resident in HBM; between timed steps L2 is flushed
              (256 MB write) -- the C5 inputs (256 MB) exceed L2 anyway.
e2e         = the same step through the public C ABI with HOST buffers:
              nestgpu_load_column from pinned host memory, exec,
              nestgpu_result_to_host into pinned host memory.
roofline    = the nested-loop kernel (the dominant kernel, >99.9 % of the
              step) against its integer-pipe bound.
cpu_baseline= the CPU oracle (oracle/) on a bounded sample of the same
              workload on this host's cores, plus the full-size closed-form
              ("unnested") CPU checker (oracle/unnested.py), timed.
side keys   = C5 '>' COUNT and '!=' MIN (1 step each), C2's 12-plan step
              (configs[1]), and C5 with every plan on the index path.

``--gpus N`` outside torchrun re-launches this script as N ranks (torchrun,
127.0.0.1); NESTGPU_DIST_BACKEND=gloo lets several ranks share one device.
"""
import argparse
import json
import os
import platform
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

ALU_LANES_PER_SM_CLK = 64   # 4 SMSPs x 16 lanes/clk (ALU pipe, rt_SMSP = 2 per warp instr)


def parse_args(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=("ours", "reference"), default="ours")
    ap.add_argument("--workload", default="C5", choices=("C5", "C2", "C1"))
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=2, help="e2e steps (at most --steps)")
    ap.add_argument("--no-side", action="store_true", help="skip the side keys (other plans, C2, index path)")
    ap.add_argument("--no-check", action="store_true", help="skip rank 0's whole-R result check")
    ap.add_argument("--gather", choices=("peer", "nccl"), default="peer",
                    help="N > 1: survivors to rank 0 by peer stores into an IPC window (default) or NCCL send/recv")
    ap.add_argument("--index-mode", choices=("local", "broadcast"), default="local",
                    help="N > 1: every rank builds the index from its resident S (default), or rank 0 builds "
                         "and broadcasts it")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="CPU oracle sample budget")
    ap.add_argument("--out", default=None, help="also append the JSON line to this file")
    return ap.parse_args(argv)


# ---------------------------------------------------------------- workloads
DESC = {
    "C5": "C5: non-equality Query 1 '>' MIN, |R|=|S|=16M int32 (col1 U[0,2^31-1), col2 U[0,2^20)), "
          "tiled nested loop",
    "C2": "C2: Query 1 family |R|=|S|=1M int32, corr op {=,<,>,!=} x agg {min,count,exists} (12 plans)",
    "C1": "C1: Query 1 |R|=|S|=1000 int32, '=' and '>' with min",
}


def workload(name):
    """(R, S, [(plan, mode)], cfg): the whole R (sharded by the caller)."""
    from datagen import make_plan, query1
    if name == "C2":
        sweep = query1.C2_SWEEP
    elif name == "C1":
        sweep = [("=", "min"), (">", "min")]
    else:
        sweep = [(">", "min")]
    cfg = dict(query1.CONFIGS[name])
    t = query1.tables(**cfg)
    plans = [(make_plan(op, agg, "="), "index" if op == "=" else "bnl") for op, agg in sweep]
    return t["R"], t["S"], plans, cfg


# ---------------------------------------------------------------- clocks
class ClockSampler:
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
               0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        self._t = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

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
            time.sleep(0.1)

    def __enter__(self):
        if self.nv:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._t:
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"]}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ---------------------------------------------------------------- CPU baselines
def cpu_model():
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return platform.processor() or "unknown"


def time_oracle(tables, plans, budget_s, calib_rows=8):
    """Time the oracle (as it stands) on a bounded sample: the first m rows of
    R for every plan, m sized to ~budget_s seconds on this host.  The size is
    found by growing a calibration sample 4x until it runs >= budget/8 (a
    handful of rows under-fills the oracle's OpenMP threads and would
    overestimate the per-row cost), then scaled to the budget."""
    import oracle
    n_r = len(tables["R"]["col1"])
    n_s = len(tables["S"]["col1"])

    def run(m):
        t0 = time.perf_counter()
        for plan, _ in plans:
            oracle.evaluate(tables, plan, rows=np.arange(m))
        return time.perf_counter() - t0

    m = min(calib_rows, n_r)
    t = run(m)
    while t < budget_s / 8 and m < n_r:
        m = min(n_r, m * 4)
        t = run(m)
    m = int(max(1, min(n_r, m * budget_s / max(t, 1e-6))))
    dt = run(m)
    for _ in range(2):   # per-call overhead makes the cost sub-linear in m: rescale until ~budget
        if dt >= budget_s / 2 or m >= n_r:
            break
        m = int(max(1, min(n_r, m * budget_s / max(dt, 1e-6))))
        dt = run(m)
    return {"value": m * len(plans) / dt, "unit": "outer tuples/s", "cores": oracle.max_threads(),
            "kind": "oracle", "seconds": dt, "cpu_model": cpu_model(), "sample_rows": m,
            "pairs_per_s": m * len(plans) * n_s / dt,
            "sample": "first %d R rows x all %d S rows for each of the %d plans (%d outer tuples)" % (
                m, n_s, len(plans), m * len(plans))}


def time_closed_form(R, S, plans):
    """The full-size closed-form 'unnested' CPU checker (oracle/unnested.py:
    sort S + prefix aggregates + binary search + outer comparison) on the
    whole workload, single-threaded numpy; outer tuples/s."""
    from oracle import unnested
    t0 = time.perf_counter()
    for plan, _ in plans:
        valid, value, cnt, s_sum = unnested.closed_form(R["col1"], S["col1"], S["col2"], plan["corr_op"], plan["agg"])
        unnested.outer_passed(R["col2"], valid, value, cnt, s_sum, plan["agg"], plan["outer_op"])
    dt = time.perf_counter() - t0
    n = len(R["col1"]) * len(plans)
    return {"value": n / dt, "unit": "outer tuples/s", "seconds": dt, "cores": 1,
            "kind": "closed-form unnested checker (sort + prefix aggregates + binary search, numpy)",
            "sample": "full workload: %d outer tuples over %d S rows" % (n, len(S["col1"]))}


def ncu_traffic(workload_name):
    """dram bytes per launch of the dominant kernel from the committed ncu
    summary (profiles/bnl_ncu_summary.json), or None."""
    path = os.path.join(ROOT, "profiles", "bnl_ncu_summary.json")
    try:
        d = json.load(open(path))
        return d.get("workloads", {}).get(workload_name, {}).get("dram_bytes_per_launch")
    except Exception:
        return None


# Pipe-bound pair rate of each nested-loop variant (pairs / clk / SM), from its
# SASS: MIN/MAX issue ISETP + predicated VIMNMX, both on
# the ALU pipe (64 lanes/clk/SM) -> 32 pairs/clk; COUNT issues ISETP (ALU) +
# predicated IMAD (FMA-heavy, 64 lanes/clk/SM) -> 64 pairs/clk; SUM/AVG (small
# payloads) ISETP + 2 predicated IMADs (FMA-heavy) -> 32 pairs/clk.
PAIRS_PER_SM_CLK = {"min": 32.0, "max": 32.0, "count": 64.0, "sum": 32.0, "avg": 32.0}
OPS_PER_PAIR = 2.0   # algorithmic: one compare + one combine per (r, s) pair


def bnl_roofline(profs, n_r, n_s, sm_max_mhz, workload_name, n_sm=148):
    """Aggregate roofline of the nested-loop kernel over the timed launches:
    frac = sum(pipe-bound time) / sum(measured time), per-launch times from
    CUDA events on the engine stream around the kernel."""
    t_act = t_ideal = ops = 0.0
    per = {}
    for plan, mode, prof, n_eval in profs:
        agg = plan["agg"]
        if mode != "bnl" or agg not in PAIRS_PER_SM_CLK:
            continue
        pairs = float(n_eval) * n_s   # outer keys evaluated (distinct ones with caching) x |S'|
        ideal = pairs / (n_sm * PAIRS_PER_SM_CLK[agg] * sm_max_mhz * 1e6)
        act = prof["subquery"] / 1000.0
        t_act += act
        t_ideal += ideal
        ops += OPS_PER_PAIR * pairs
        d = per.setdefault(agg, {"launches": 0, "ms": 0.0, "ideal_ms": 0.0})
        d["launches"] += 1
        d["ms"] += act * 1000
        d["ideal_ms"] += ideal * 1000
    if not t_act:
        return None
    for d in per.values():
        d["frac"] = d["ideal_ms"] / d["ms"]
        d["ms_per_launch"] = d["ms"] / d["launches"]
    return {"bound": "alu", "achieved": ops / t_act / 1e12, "peak": ops / t_ideal / 1e12, "unit": "Tops/s",
            "frac": t_ideal / t_act, "traffic": ncu_traffic(workload_name),
            "kernel": "bnl_kernel (tiled block-nested loop)",
            "algorithmic": "2 integer ops (compare + combine) per (r,s) pair x |R'| x |S'| per launch",
            "peak_source": ("integer pipes: %d SMs x %.0f MHz (sm_max_mhz, MEASURED_PEAKS.json) x "
                            "ALU 64 lanes/clk (MIN: 2 ALU ops/pair) | ALU+FMA-heavy 64 lanes/clk each "
                            "(COUNT: 1+1 ops/pair); B300_MICROARCH pipe rates" % (n_sm, sm_max_mhz)),
            "per_agg": per}


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def emit(line, args):
    s = json.dumps(line)
    print(s, flush=True)
    if args.out:
        with open(args.out, "a") as f:
            f.write(s + "\n")


# ---------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    """The oracle, as it stands, on the host cores: each step a bounded sample
    of the workload.  Under torchrun only rank 0 works."""
    if rank != 0:
        return
    R, S, plans, cfg = workload(args.workload)
    tables = {"R": R, "S": S}
    per_step = max(1.0, args.cpu_seconds / 2.0)
    for _ in range(args.warmup):
        time_oracle(tables, plans, per_step / 4)
    vals, secs = [], []
    cb = None
    for _ in range(args.steps):
        cb = time_oracle(tables, plans, per_step)
        vals.append(cb["value"])
        secs.append(cb["seconds"])
    value = statistics.median(vals)
    line = {"metric": "outer tuples/s", "value": value, "unit": "outer tuples/s", "impl": "reference",
            "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000 * statistics.median(secs), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "int64", "data": "synthetic (seeded in-repo generator)",
            "config": {"workload": DESC[args.workload], "n_r": cfg["n_r"], "n_s": cfg["n_s"],
                       "plans": len(plans), "sampled": True},
            "cpu_baseline": {"value": value, "unit": "outer tuples/s", "cores": cb["cores"], "kind": "oracle",
                             "cpu_model": cb["cpu_model"], "sample": cb["sample"]},
            "e2e": {"value": value, "unit": "outer tuples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line, args)


# ---------------------------------------------------------------- our arm
class Rank:
    """One rank's engine state for one workload: its R shard (resident), S
    (broadcast from rank 0 at N > 1, resident) and the step function."""

    def __init__(self, eng, dev, stream, name, rank, world, R, S, plans, gather="peer", index_mode="local"):
        from paper_conf_icde_floratosxwgylz21_b200 import dist as ngd
        self.ngd = ngd
        self.gather_mode, self.index_mode = gather, index_mode
        self.eng, self.dev, self.stream = eng, dev, stream
        self.name, self.rank, self.world = name, rank, world
        self.R_full, self.S_host, self.plans = R, S, plans
        self.n_r, self.n_s = len(R["col1"]), len(S["col1"])
        self.lo, self.hi = ngd.shard_range(self.n_r, rank, world)
        self.R_shard = {k: np.ascontiguousarray(v[self.lo:self.hi]) for k, v in R.items()}
        self.Rc = eng.load_table(self.R_shard)
        if world > 1:
            self.Sc = ngd.share_table(eng, S if rank == 0 else None, list(S), self.n_s, device=dev)
        else:
            self.Sc = eng.load_table(S)
        self.launches = 0
        self.pg = None
        self.gather_note = None
        if world > 1 and gather == "peer":
            self.pg = ngd.PeerGather(eng, self.n_r, device=dev)
            if not self.pg.ok:   # some rank cannot map rank 0's window: NCCL send/recv instead
                self.gather_note = "peer window unavailable (%s); NCCL send/recv used" % self.pg.error
                self.pg = None

    def step(self, plans=None, profs=None, stages=None, keep=None):
        """One pass of the hot path over the batch (every plan).  At N > 1 the
        index (if a plan needs one) is built on rank 0 and broadcast, and each
        plan's survivors are gathered to rank 0.  keep: list that receives the
        per-plan survivors (rank 0; (rows, values) torch tensors)."""
        import torch
        eng, ngd = self.eng, self.ngd
        plans = self.plans if plans is None else plans
        m = eng.mark()
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(2 + 2 * len(plans))] if stages is not None else None
        if ev:
            ev[0].record(self.stream)
        idx = {}
        for plan, mode in plans:
            if mode == "index":
                payload = "col2" if plan["agg"] in ("min", "max", "sum", "avg") else None
                if payload not in idx:
                    idx[payload] = (ngd.share_index(eng, self.Sc, ["col1"], payload, device=self.dev)
                                    if self.world > 1 and self.index_mode == "broadcast"
                                    else eng.build_index(self.Sc, ["col1"], payload))
        if ev:
            ev[1].record(self.stream)
        out = []
        for i, (plan, mode) in enumerate(plans):
            payload = "col2" if plan["agg"] in ("min", "max", "sum", "avg") else None
            res = eng.exec(plan, self.Rc, self.Sc, index=idx[payload] if mode == "index" else -1,
                           row_id_base=self.lo)
            if ev:
                ev[2 + 2 * i].record(self.stream)
            if profs is not None:
                profs.append((plan, mode, eng.last_profile(), res.n_evaluated))
            out.append(res.n_rows)
            if self.world > 1:
                if self.pg is not None:
                    g = self.pg.gather(res)
                else:
                    t = eng.result_tensors(res)
                    g = ngd.gather_rows([t["row"], t["value"]])
                if keep is not None and self.rank == 0:
                    keep.append((g[0].clone(), g[1].clone()))
            elif keep is not None:
                t = eng.result_tensors(res)
                keep.append((t["row"].clone(), t["value"].clone()))
            if ev:
                ev[3 + 2 * i].record(self.stream)
        eng.release(m)
        if ev:
            ev[-1].synchronize()
            stages["index_build_broadcast"] = stages.get("index_build_broadcast", 0.0) + ev[0].elapsed_time(ev[1])
            ex = ga = 0.0
            prev = ev[1]
            for i in range(len(plans)):
                ex += prev.elapsed_time(ev[2 + 2 * i])
                ga += ev[2 + 2 * i].elapsed_time(ev[3 + 2 * i])
                prev = ev[3 + 2 * i]
            stages["exec"] = stages.get("exec", 0.0) + ex
            stages["gather"] = stages.get("gather", 0.0) + ga
        return out

    def timed(self, k, flush, plans=None, profs=None, stages=None, keep_last=None):
        """k steps, each bracketed by CUDA events on the engine stream, L2
        flushed before each; returns per-step ms (this rank)."""
        import torch
        ms = []
        for i in range(k):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(self.stream)
            keep = [] if (keep_last is not None and i == k - 1) else None
            self.step(plans, profs, stages, keep)
            e1.record(self.stream)
            e1.synchronize()
            ms.append(e0.elapsed_time(e1))
            if keep is not None:
                keep_last[:] = keep
        return ms

    def check_whole_r(self, plans, gathered):
        """Rank 0: the whole-R result of each plan on the 1-GPU index path
        (sorted index + binary search / prefix aggregates -- a different
        kernel from the nested loop), compared with the gathered survivors.
        Returns a dict, or None on other ranks."""
        if self.rank != 0:
            return None
        import torch
        eng = self.eng
        m = eng.mark()
        Rw = eng.load_table(self.R_full) if self.world > 1 else self.Rc
        ok, n_cmp = True, 0
        for (plan, _), (rows, vals) in zip(plans, gathered):
            payload = "col2" if plan["agg"] in ("min", "max", "sum", "avg") else None
            idx = eng.build_index(self.Sc, ["col1"], payload)
            res = eng.exec(plan, Rw, self.Sc, index=idx)
            t = eng.result_tensors(res)
            same = (t["row"].numel() == rows.numel() and bool(torch.equal(t["row"], rows))
                    and bool(torch.equal(t["value"], vals)))
            ok = ok and same
            n_cmp += int(rows.numel())
        eng.release(m)
        return {"identical": ok, "plans": len(plans), "survivors_compared": n_cmp,
                "reference": "whole R on 1 GPU, index path (sorted index + prefix aggregates)"}


def main(argv=None):
    args = parse_args(argv)
    in_env = "WORLD_SIZE" in os.environ
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)
    if args.gpus > 1 and not in_env:
        from paper_conf_icde_floratosxwgylz21_b200 import dist as ngd
        return ngd.launch_ranks(os.path.abspath(__file__), list(sys.argv[1:] if argv is None else argv), args.gpus)

    import torch
    import torch.distributed as dist
    from paper_conf_icde_floratosxwgylz21_b200 import Engine, dist as ngd

    dev_idx = local_rank % max(1, torch.cuda.device_count())
    torch.cuda.set_device(dev_idx)
    dev = torch.device("cuda", dev_idx)
    backend = ngd.backend_name() if world > 1 else None
    nccl_pat = None
    if world > 1:
        if backend == "nccl":
            nccl_pat = ngd.nccl_debug_setup()
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)

    R, S_host, plans, cfg = workload(args.workload)
    n_r, n_s = len(R["col1"]), len(S_host["col1"])
    arena = max(1 << 30, (n_r + n_s) * 8 * 24 + (512 << 20))
    eng = Engine(dev_idx, arena_bytes=arena, stream=stream)
    eng.set_profiling(True)
    rk = Rank(eng, dev, stream, args.workload, rank, world, R, S_host, plans, args.gather, args.index_mode)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        rk.step()
    barrier()

    # ---- timed region: K steps
    profs, stages, last = [], {}, []
    launches0 = eng.launch_count()
    with ClockSampler(dev_idx) as clocks:
        step_ms = rk.timed(args.steps, flush, profs=profs, stages=stages, keep_last=last)
    torch.cuda.synchronize()
    launches = ngd.sum_over_ranks(eng.launch_count() - launches0, device=dev) if world > 1 else \
        eng.launch_count() - launches0
    barrier()
    total_ms = ngd.max_over_ranks(sum(step_ms), device=dev)
    ms_per_step = total_ms / args.steps
    outer_per_step = len(plans) * n_r
    value = outer_per_step / (ms_per_step / 1000.0)
    surv = [int(r.numel()) for r, _ in last] if rank == 0 else []

    pk = peaks()
    sm_max = pk.get("sm_max_mhz") or clocks.summary().get("sm_max_mhz") or 1965.0
    n_eval_shard = rk.hi - rk.lo
    roofline = bnl_roofline(profs, n_eval_shard, n_s, sm_max, args.workload)
    eng_stages = {}
    for _, _, prof, _ in profs:
        for k, v in prof.items():
            if v == v:  # not NaN
                eng_stages[k] = eng_stages.get(k, 0.0) + v / args.steps
    multi = {k: v / args.steps for k, v in stages.items()}

    # ---- T7: N-GPU survivors == the 1-GPU whole-R result (another kernel)
    check = None
    if not args.no_check:
        check = rk.check_whole_r(plans, last)
        barrier()

    # ---- side keys (not the headline; 1 step each, all ranks)
    side = {}
    if not args.no_side:
        from datagen import make_plan
        if args.workload == "C5":
            for op, agg in ((">", "count"), ("!=", "min")):
                sp = [(make_plan(op, agg, "="), "bnl")]
                sprof, skeep = [], []
                ms = rk.timed(1, flush, plans=sp, profs=sprof, keep_last=skeep)
                t = ngd.max_over_ranks(sum(ms), device=dev)
                rf = bnl_roofline(sprof, n_eval_shard, n_s, sm_max, args.workload)
                chk = None if args.no_check else rk.check_whole_r(sp, skeep)
                barrier()
                side["%s %s (nested loop)" % (op, agg)] = {
                    "value": n_r / (t / 1000.0), "ms_per_step": t, "steps": 1,
                    "roofline_frac": rf["frac"] if rf else None,
                    "survivors": int(skeep[0][0].numel()) if (rank == 0 and skeep) else None,
                    "check": chk}
        # every plan on the index path (index-pruned evaluation, NEXT 3)
        ip = [(p, "index") for p, _ in plans]
        rk.step(ip)
        barrier()
        ms = rk.timed(max(1, min(args.steps, 5)), flush, plans=ip)
        t = ngd.max_over_ranks(sum(ms), device=dev) / len(ms)
        side["index_pruned (all plans on the index path)"] = {
            "value": outer_per_step / (t / 1000.0), "ms_per_step": t, "steps": len(ms),
            "note": "sorted index built every step (on every rank; broadcast from rank 0 with "
                    "--index-mode broadcast) + binary search; non-equality ranges from prefix/suffix aggregates"}
        if args.workload == "C5":
            # C2's 12-plan step (BASELINE configs[1]) as an extra key
            R2, S2, plans2, _ = workload("C2")
            m0 = eng.mark()
            rk2 = Rank(eng, dev, stream, "C2", rank, world, R2, S2, plans2, args.gather, args.index_mode)
            for _ in range(2):
                rk2.step()
            barrier()
            k2 = max(3, min(args.steps, 10))
            prof2 = []
            ms = rk2.timed(k2, flush, profs=prof2)
            t = ngd.max_over_ranks(sum(ms), device=dev) / k2
            rf2 = bnl_roofline(prof2, rk2.hi - rk2.lo, len(S2["col1"]), sm_max, "C2")
            side["C2 12-plan step"] = {"value": len(plans2) * len(R2["col1"]) / (t / 1000.0), "ms_per_step": t,
                                       "steps": k2, "workload": DESC["C2"],
                                       "roofline_frac": rf2["frac"] if rf2 else None}
            if rk2.pg is not None:
                rk2.pg.close()
            del rk2
            eng.release(m0)
            barrier()

    # ---- e2e through the public API with host buffers (pinned), every step
    e2e = None
    if not args.no_e2e:
        pin = {k: torch.from_numpy(v).pin_memory() for k, v in rk.R_shard.items()}
        pin_s = {k: torch.from_numpy(np.ascontiguousarray(v)).pin_memory() for k, v in S_host.items()}
        h2d = sum(v.numel() * v.element_size() for v in pin.values()) + sum(
            v.numel() * v.element_size() for v in pin_s.values())
        nloc = rk.hi - rk.lo if world == 1 or rank != 0 else n_r   # rank 0 receives every rank's survivors
        res_pin = {k: torch.empty(max(1, nloc), dtype=dt, pin_memory=True).numpy()
                   for k, dt in (("row", torch.int64), ("value", torch.int64), ("valid", torch.uint8),
                                 ("passed", torch.uint8))}
        d2h = [0]

        def e2e_step():
            m = eng.mark()
            Rx = {k: eng.load_column(v) for k, v in pin.items()}
            Sx = {k: eng.load_column(v) for k, v in pin_s.items()}
            idx = {}
            nb = 0
            for plan, mode in plans:
                payload = "col2" if plan["agg"] in ("min", "max", "sum", "avg") else None
                if mode == "index" and payload not in idx:
                    idx[payload] = eng.build_index(Sx, ["col1"], payload)
                res = eng.exec(plan, Rx, Sx, index=idx[payload] if mode == "index" else -1, row_id_base=rk.lo)
                if world > 1:   # the survivors reach rank 0 (window / NCCL), then rank 0's host
                    if rk.pg is not None:
                        g = rk.pg.gather(res)
                    else:
                        t = eng.result_tensors(res)
                        g = ngd.gather_rows([t["row"], t["value"]])
                    if rank == 0:
                        n_g = int(g[0].numel())
                        res_pin["row"][:n_g] = g[0].cpu().numpy()
                        res_pin["value"][:n_g] = g[1].cpu().numpy()
                        nb += 16 * n_g
                else:
                    out = eng.result_to_numpy(res, out=res_pin)
                    nb += sum(a.nbytes for a in out.values())
            eng.release(m)
            d2h[0] = nb

        ke = max(1, min(args.steps, args.e2e_steps))
        e2e_step()
        barrier()
        e2e_ms = []
        for _ in range(ke):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            e2e_step()
            e1.record(stream)
            e1.synchronize()
            e2e_ms.append(e0.elapsed_time(e1))
        e2e_t = ngd.max_over_ranks(sum(e2e_ms), device=dev) / ke
        e2e = {"value": outer_per_step / (e2e_t / 1000.0), "unit": "outer tuples/s", "ms_per_step": e2e_t,
               "steps": ke,
               "h2d_bytes_per_step": int(ngd.sum_over_ranks(h2d, device=dev) if world > 1 else h2d),
               "d2h_bytes_per_step": int(ngd.sum_over_ranks(d2h[0], device=dev) if world > 1 else d2h[0]),
               "path": ("nestgpu_load_column (pinned host) -> [build_index] -> exec x%d -> "
                        "nestgpu_result_to_host (pinned host)" % len(plans)) if world == 1 else
                       ("per rank: nestgpu_load_column (pinned host) -> [build_index] -> exec x%d -> survivors "
                        "gathered to rank 0 (%s) -> rank 0 host" % (len(plans), args.gather))}

    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline:
            cpu = time_oracle({"R": R, "S": S_host}, plans, args.cpu_seconds)
            cpu["closed_form"] = time_closed_form(R, S_host, plans)
        latency = {}
        for plan, mode, prof, _ in profs:
            key = "%s %s (%s)" % (plan["corr_op"], plan["agg"], mode)
            latency.setdefault(key, []).append(prof["total"])
        par = "1 GPU" if world == 1 else (
            "R sharded x%d (contiguous row blocks, one R), S broadcast once (%s), index %s, survivors gathered "
            "to rank 0 each step by %s" % (
                world, backend, "built on every rank" if args.index_mode == "local" else "built on rank 0 + broadcast",
                "peer stores into an IPC window on rank 0" if args.gather == "peer" else "NCCL send/recv"))
        line = {
            "metric": "outer tuples/s", "value": value, "unit": "outer tuples/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic (seeded in-repo Query-1 generator, datagen/query1.py)",
            "config": {"workload": DESC[args.workload], "n_r": n_r, "n_s": n_s, "n_r_per_gpu": n_r / world,
                       "plans": len(plans), "pairs_per_step": float(len(plans)) * n_r * n_s,
                       "index_path": "'=' plans", "nested_loop_path": "'<','>','!=' plans",
                       "l2": "flushed between timed steps (256 MB write); inputs %d MB" % (
                           (n_r + n_s) * 8 >> 20),
                       "parallelism": par},
            "roofline": roofline,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": int(launches),
            "clocks": clocks.summary(),
            "query_latency_ms": {k: statistics.median(v) for k, v in latency.items()},
            "stages_ms_per_step": eng_stages,
            "multi_gpu_stages_ms_per_step": multi if world > 1 else None,
            "survivors_per_plan": surv,
            "whole_r_check": check,
            "side": side,
            "step_ms": step_ms,
        }
        if nccl_pat:
            line["nccl_init"] = ngd.nccl_init_summary(nccl_pat)
        if rk.gather_note:
            line["gather_note"] = rk.gather_note
        emit(line, args)
    if rk.pg is not None:
        rk.pg.close()
    eng.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main() or 0)
