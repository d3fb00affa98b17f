#!/usr/bin/env python
"""Benchmark of the nested-method correlated-subquery hot path on B200.

Metric (BASELINE.json): outer tuples/s (+ query latency, roofline fraction).
Workload: BASELINE.json configs[1] ("C2") -- the Query 1 family
(PAPER.md P:41 / P:53) at |R| = |S| = 1M, correlated operator sweep
{=, <, >, !=} x aggregate sweep {min, count, exists} = 12 plans.  One step
is one pass of the whole hot path over that batch:

  build the correlated-column index of S (filter + radix sort; the paper
  includes index build in its timings), then for each plan: outer
  filter -> subquery kernel (index range-aggregate for '=', tiled nested
  loop for '<', '>', '!=') -> aggregate finalize + outer comparison ->
  compaction of the survivors.

value       = outer tuples evaluated per second over all ranks
              (12 plans x |R| per rank x ranks / step time), inputs resident
              in HBM, L2 flushed (256 MB write) between timed steps.
e2e         = the same through the public C ABI with HOST buffers: every step
              copies R and S from pinned host memory (nestgpu_load_column) and
              reads every survivor back (nestgpu_result_to_host).
roofline    = the nested-loop kernel (the dominant kernel) against the
              integer-ALU pipe peak.
cpu_baseline= the CPU oracle (oracle/) timed on a bounded sample of the same
              plans on this host's cores.

Multi-GPU (torchrun): R is sharded (|R| = 1M per rank, weak scaling), rank 0
builds the index and broadcasts it over NCCL into every rank's arena each
step; survivors are gathered to rank 0 each step.
"""
import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

ALU_LANES_PER_SM_CLK = 64   # 4 SMSPs x 16 lanes/clk (ALU pipe, rt_SMSP = 2 per warp instr)


def parse_args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=("ours", "reference"), default="ours")
    ap.add_argument("--workload", default="C2", choices=("C2", "C1", "C5"))
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--dedup", action="store_true",
                    help="headline with P:331 caching (one subquery evaluation per distinct correlated value)")
    ap.add_argument("--no-variants", action="store_true", help="skip the with/without-caching side measurement")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="CPU oracle sample budget")
    ap.add_argument("--out", default=None, help="also append the JSON line to this file")
    return ap.parse_args()


# ---------------------------------------------------------------- workload
def workload(name, rank):
    from datagen import make_plan, query1
    if name == "C2":
        sweep = query1.C2_SWEEP
        cfg = dict(query1.CONFIGS["C2"])
    elif name == "C1":
        sweep = [("=", "min"), (">", "min")]
        cfg = dict(query1.CONFIGS["C1"])
    else:  # C5: non-equality Query 1 at 16M
        sweep = [(">", "min")]
        cfg = dict(query1.CONFIGS["C5"])
    t0 = query1.tables(**cfg)                       # rank 0's R and the shared S
    if rank == 0:
        R = t0["R"]
    else:                                           # weak scaling: a fresh R block per rank
        R = query1.tables(**dict(cfg, seed=cfg["seed"] + 1000 * rank))["R"]
    plans = [(make_plan(op, agg, "="), "index" if op == "=" else "bnl") for op, agg in sweep]
    desc = {
        "C2": "Query 1 family |R|=|S|=1M int32, corr op {=,<,>,!=} x agg {min,count,exists} (12 plans)",
        "C1": "Query 1 |R|=|S|=1000 int32, '=' and '>' with min",
        "C5": "non-equality Query 1 '>' min, |R|=|S|=16M int32",
    }[name]
    return R, t0["S"], plans, desc, cfg


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


# ---------------------------------------------------------------- CPU oracle
def time_oracle(tables, plans, budget_s, calib_rows=8):
    """Time the oracle (as it stands) on a bounded sample: the first m rows of
    R for every plan, m sized to ~budget_s seconds on this host.  The size is
    found by growing a calibration sample 4x until it runs >= budget/8 (a
    handful of rows under-fills the oracle's OpenMP threads and would
    overestimate the per-row cost), then scaled to the budget."""
    import oracle
    n_r = len(tables["R"]["col1"])

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
            "kind": "oracle", "seconds": dt,
            "sample": "first %d R rows x all %d S rows for each of the %d plans (%d outer tuples)" % (
                m, len(tables["S"]["col1"]), len(plans), m * len(plans))}


def ncu_traffic(workload_name):
    """dram bytes per launch of the dominant kernel from the committed ncu
    --set full summary (profiles/), or None."""
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


def bnl_roofline(profs, n_r, n_s, sm_max_mhz, workload_name):
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
        ideal = pairs / (148 * PAIRS_PER_SM_CLK[agg] * sm_max_mhz * 1e6)
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
            "kernel": "bnl_kernel (tiled block-nested loop), MIN and COUNT launches",
            "algorithmic": "2 integer ops (compare + combine) per (r,s) pair x |R'| x |S'| per launch",
            "peak_source": ("integer pipes: 148 SMs x %.0f MHz (sm_max_mhz, MEASURED_PEAKS.json) x "
                            "ALU 64 lanes/clk (MIN: 2 ALU ops/pair) | ALU+FMA-heavy 64 lanes/clk each "
                            "(COUNT: 1+1 ops/pair); B300_MICROARCH pipe rates" % sm_max_mhz),
            "per_agg": per}


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


# ---------------------------------------------------------------- reference arm
def run_reference(args, rank, world):
    if rank != 0:
        return
    R, S, plans, desc, cfg = workload(args.workload, 0)
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
            "ms_per_step": 1000 * statistics.median(secs), "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int64", "data": "synthetic (seeded in-repo generator)",
            "config": {"workload": args.workload + ": " + desc, "n_r": cfg["n_r"], "n_s": cfg["n_s"],
                       "plans": len(plans), "sampled": True},
            "cpu_baseline": {"value": value, "unit": "outer tuples/s", "cores": cb["cores"], "kind": "oracle",
                             "sample": cb["sample"]},
            "e2e": {"value": value, "unit": "outer tuples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    emit(line, args)


def emit(line, args):
    s = json.dumps(line)
    print(s, flush=True)
    if args.out:
        with open(args.out, "a") as f:
            f.write(s + "\n")


# ---------------------------------------------------------------- our arm
def main():
    args = parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import torch
    import torch.distributed as dist
    from paper_conf_icde_floratosxwgylz21_b200 import Engine, dist as ngd

    # one process per GPU (NCCL); NESTGPU_DIST_BACKEND=gloo lets several ranks
    # share one device for functional runs of the multi-rank path
    dev_idx = local_rank % max(1, torch.cuda.device_count())
    torch.cuda.set_device(dev_idx)
    dev = torch.device("cuda", dev_idx)
    if world > 1:
        if ngd.backend_name() == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(ngd.backend_name())
    R, S_host, plans, desc, cfg = workload(args.workload, rank)
    n_r, n_s = len(R["col1"]), len(S_host["col1"])
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)
    need = (n_r + n_s) * 8 * 16 + (256 << 20)
    eng = Engine(dev_idx, arena_bytes=max(need, 1 << 30), stream=stream)

    # ---- resident inputs (untimed): R shard per rank, S on rank 0 then broadcast
    Rc = eng.load_table(R)
    if world > 1:
        Sc = ngd.share_table(eng, S_host if rank == 0 else None, ["col1", "col2"], n_s, device=dev)
    else:
        Sc = eng.load_table(S_host)
    base_mark = eng.mark()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    row_base = ngd.shard_range(n_r * world, rank, world)[0]

    def step(profile_sink=None, dedup=args.dedup):
        """One pass of the hot path over the batch (all plans)."""
        m = eng.mark()
        need_index = any(mode == "index" for _, mode in plans)
        idx = -1
        if need_index:   # rank 0 sorts; the index is broadcast to the other ranks
            idx = (ngd.share_index(eng, Sc, ["col1"], "col2", device=dev) if world > 1
                   else eng.build_index(Sc, ["col1"], "col2"))
        surv = []
        evals.clear()
        gathered = []
        for plan, mode in plans:
            res = eng.exec(plan, Rc, Sc, index=idx if mode == "index" else -1, row_id_base=row_base, dedup=dedup)
            surv.append(res.n_rows)
            evals.append(res.n_evaluated)
            if profile_sink is not None:
                profile_sink.append((plan, mode, eng.last_profile(), res.n_evaluated))
            if world > 1:
                t = eng.result_tensors(res)
                gathered.append((t["row"].clone(), t["value"].clone()))
        if world > 1:
            rows = torch.cat([g[0] for g in gathered])
            vals = torch.cat([g[1] for g in gathered])
            ngd.gather_rows([rows, vals])
        eng.release(m)
        return surv

    evals = []
    eng.set_profiling(True)
    for _ in range(args.warmup):
        step()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()

    # ---- timed region: K steps, per-step CUDA events on the engine stream, L2 flushed between
    step_ms, profs = [], []
    launches0 = eng.launch_count()
    with ClockSampler(local_rank) as clocks:
        for _ in range(args.steps):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            surv = step(profs)
            e1.record(stream)
            e1.synchronize()
            step_ms.append(e0.elapsed_time(e1))
    torch.cuda.synchronize()
    launches = eng.launch_count() - launches0
    evals_main = list(evals)
    if world > 1:
        dist.barrier()
    total_ms = ngd.max_over_ranks(sum(step_ms), device=dev)
    ms_per_step = total_ms / args.steps
    outer_per_step = len(plans) * n_r * world
    value = outer_per_step / (ms_per_step / 1000.0)

    # ---- dominant kernel: the nested loop (min / count plans; EXISTS stops early)
    pk = peaks()
    sm_max = pk.get("sm_max_mhz") or clocks.summary().get("sm_max_mhz") or 1965.0
    roofline = bnl_roofline(profs, n_r, n_s, sm_max, args.workload)
    stages = {}
    for _, _, prof, _ in profs:
        for k, v in prof.items():
            if v == v:  # not NaN
                stages[k] = stages.get(k, 0.0) + v / args.steps

    # ---- side measurements (not the headline): the same step with the other
    # caching setting, and with every plan on the index path
    # (index-pruned evaluation).
    def time_steps(fn, k):
        ms = []
        for _ in range(k):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            e1.synchronize()
            ms.append(e0.elapsed_time(e1))
        return ngd.max_over_ranks(sum(ms), device=dev) / len(ms)

    variant = None
    index_variant = None
    if not args.no_variants:
        v_ms = time_steps(lambda: step(dedup=not args.dedup), max(1, args.steps))
        variant = {"dedup": not args.dedup, "value": outer_per_step / (v_ms / 1000.0), "ms_per_step": v_ms,
                   "subquery_evaluations_per_plan": list(evals)}
        saved = list(plans)
        plans[:] = [(p, "index") for p, _ in saved]
        step()
        i_ms = time_steps(step, max(1, args.steps))
        plans[:] = saved
        index_variant = {"all_plans_on_index_path": True, "value": outer_per_step / (i_ms / 1000.0),
                         "ms_per_step": i_ms,
                         "note": "sorted index + binary search; non-equality ranges from prefix/suffix aggregates"}

    # ---- e2e through the public API with host buffers
    e2e = None
    if not args.no_e2e:
        pin = {k: torch.from_numpy(np.ascontiguousarray(v)).pin_memory() for k, v in R.items()}
        pin_s = {k: torch.from_numpy(np.ascontiguousarray(v)).pin_memory() for k, v in S_host.items()}
        h2d = sum(v.numel() * v.element_size() for v in pin.values()) + sum(
            v.numel() * v.element_size() for v in pin_s.values())
        eng.release(base_mark)
        e2e_ms, d2h = [], 0

        # result buffers: pinned host memory allocated once, reused every step
        # (like the pinned inputs); sized for every R row of one plan
        res_pin = {k: torch.empty(n_r, dtype=dt, pin_memory=True).numpy()
                   for k, dt in (("row", torch.int64), ("value", torch.int64), ("valid", torch.uint8),
                                 ("passed", torch.uint8))}

        def e2e_step():
            nonlocal d2h
            m = eng.mark()
            Rx = {k: eng.load_column(v) for k, v in pin.items()}
            Sx = {k: eng.load_column(v) for k, v in pin_s.items()}
            idx = eng.build_index(Sx, ["col1"], "col2") if any(md == "index" for _, md in plans) else -1
            nb = 0
            for plan, mode in plans:
                res = eng.exec(plan, Rx, Sx, index=idx if mode == "index" else -1, row_id_base=row_base,
                           dedup=args.dedup)
                out = eng.result_to_numpy(res, out=res_pin)
                nb += sum(a.nbytes for a in out.values())
            eng.release(m)
            d2h = nb

        for _ in range(max(1, args.warmup // 2)):
            e2e_step()
        torch.cuda.synchronize()
        for _ in range(args.steps):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            e2e_step()
            e1.record(stream)
            e1.synchronize()
            e2e_ms.append(e0.elapsed_time(e1))
        e2e_t = ngd.max_over_ranks(sum(e2e_ms), device=dev) / args.steps
        e2e = {"value": outer_per_step / (e2e_t / 1000.0), "unit": "outer tuples/s", "ms_per_step": e2e_t,
               "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
               "path": "nestgpu_load_column (pinned host) -> build_index -> exec x%d -> result_to_host (pinned host)"
                       % len(plans)}

    if rank == 0:
        cpu = None
        if not args.no_cpu_baseline:
            cpu = time_oracle({"R": R, "S": S_host}, plans, args.cpu_seconds)
        latency = {}
        for plan, mode, prof, _ in profs:
            key = "%s %s (%s)" % (plan["corr_op"], plan["agg"], mode)
            latency.setdefault(key, []).append(prof["total"])
        line = {
            "metric": "outer tuples/s", "value": value, "unit": "outer tuples/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic (seeded in-repo Query-1 generator, datagen/query1.py)",
            "config": {"workload": args.workload + ": " + desc, "n_r_per_gpu": n_r, "n_s": n_s,
                       "plans": len(plans), "index_path": "'=' plans", "nested_loop_path": "'<','>','!=' plans",
                       "l2": "flushed between timed steps (256 MB write); inputs 16 MB < L2",
                       "parallelism": "R sharded x%d, index broadcast (NCCL)" % world if world > 1 else "1 GPU"},
            "roofline": roofline,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clocks.summary(),
            "query_latency_ms": {k: statistics.median(v) for k, v in latency.items()},
            "stages_ms_per_step": stages,
            "survivors_per_plan": surv,
            "dedup": args.dedup,
            "subquery_evaluations_per_plan": evals_main,
            "variant": variant,
            "variant_index_pruned": index_variant,
            "step_ms": step_ms,
        }
        emit(line, args)
    eng.close()
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
