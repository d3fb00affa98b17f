"""CPU checks of bench.py: the reference arm end to end (it times the CPU
oracle, no GPU involved) and the roofline arithmetic."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_reference_arm_prints_one_json_line():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                        "--warmup", "0", "--workload", "C1", "--cpu-seconds", "0.3"],
                       capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["metric"] == "outer tuples/s" and d["value"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["cpu_baseline"]["kind"] == "oracle"


def test_bnl_roofline_arithmetic():
    from datagen import make_plan
    n = 1_000_000
    # a MIN launch exactly at the ALU bound and a COUNT launch at half its bound
    t_min = n * n / (148 * 32 * 1965e6) * 1000
    t_cnt = 2 * n * n / (148 * 64 * 1965e6) * 1000
    profs = [(make_plan(">", "min", "="), "bnl", {"subquery": t_min}, n),
             (make_plan(">", "count", "="), "bnl", {"subquery": t_cnt}, n),
             (make_plan("=", "min", "="), "index", {"subquery": 0.1}, n)]
    r = bench.bnl_roofline(profs, n, n, 1965.0, "C2")
    ideal = t_min + t_cnt / 2
    assert abs(r["frac"] - ideal / (t_min + t_cnt)) < 1e-9
    assert abs(r["per_agg"]["min"]["frac"] - 1.0) < 1e-9
    assert abs(r["per_agg"]["count"]["frac"] - 0.5) < 1e-9
    assert r["bound"] == "alu" and abs(r["achieved"] / r["peak"] - r["frac"]) < 1e-9


import pytest  # noqa: E402


@pytest.mark.gpu
def test_bench_our_arm_c1_json_contract():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--workload", "C1", "--steps", "3",
                        "--warmup", "3", "--cpu-seconds", "0.5"], capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
              "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e", "gpu_launches", "clocks"):
        assert k in d, k
    assert d["value"] > 0 and d["gpu_launches"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0
    assert d["roofline"]["bound"] == "alu" and 0 < d["roofline"]["frac"]


@pytest.mark.gpu
def test_bench_spawns_two_ranks_gloo():
    """`bench.py --gpus 2` outside torchrun launches 2 ranks itself (here gloo,
    both on the one B200); rank 0 reports n_gpus 2 and finds the gathered
    survivors identical to the whole-R 1-GPU result."""
    env = dict(os.environ, NESTGPU_DIST_BACKEND="gloo")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--workload", "C1",
                        "--steps", "3", "--warmup", "3", "--no-cpu-baseline"], capture_output=True, text=True,
                       timeout=900, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong"
    assert d["whole_r_check"]["identical"] is True
    assert d["multi_gpu_stages_ms_per_step"]["gather"] >= 0


def test_bench_defaults_to_c5_headline():
    """The driver's `bench.py --gpus 1 --steps 20 --warmup 5` measures C5
    (BASELINE configs[4], the largest single-GPU config) -- VERDICT r1 item 1."""
    a = bench.parse_args(["--gpus", "1", "--steps", "20", "--warmup", "5"])
    assert a.workload == "C5" and a.gather == "peer" and a.index_mode == "local"
    assert bench.DESC["C5"].startswith("C5: non-equality Query 1 '>' MIN, |R|=|S|=16M")


def test_cpu_baselines_report_model_and_closed_form():
    """cpu_baseline fields: the oracle sample with the CPU model, and the
    timed closed-form checker over the whole (here C1) workload."""
    R, S, plans, _ = bench.workload("C1")
    cb = bench.time_oracle({"R": R, "S": S}, plans, 0.2)
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["cpu_model"] and cb["value"] > 0
    cf = bench.time_closed_form(R, S, plans)
    assert cf["value"] > 0 and cf["sample"].startswith("full workload: 2000 outer tuples")
