"""The cost model (§IV, Eqs. (1)-(9)): host arithmetic on CPU
(nestgpu_cost_estimate_plan needs no device), calibration + strategy choice
on the GPU.

CPU tests check the structure the paper gives the model, not a retyping of
the formulas: the vectorised per-evaluation term scales with the number of
evaluations S - Ch (Eq. (6)) and caching shrinks exactly that term; the
invariant parts (index build, S' selection) do not depend on |R'|; the
launch constant C is charged per launch, not per outer tuple (vectorisation,
P:317); the choice is the argmin; bad inputs are rejected.
"""
import math

import pytest

from paper_conf_icde_floratosxwgylz21_b200 import cost_estimate, STRATEGIES
from paper_conf_icde_floratosxwgylz21_b200.binding import NestGPUError

P = {"launch_ms": 0.003, "filter_ms_per_row": 7e-9, "hist_ms_per_key_digit": 1e-9, "sort_ms_per_key": 5e-9,
     "sort_ms_per_byte": 8e-10, "probe_ms_per_step": 5e-10, "range_ms_per_elem": 3e-10, "aux_ms_per_elem": 2e-8,
     "bnl_ms_per_pair": [[1.1e-10, 7e-11, 1.3e-10, 6e-11], [2.2e-10, 1.4e-10, 2.6e-10, 1.2e-10]],
     "final_ms_per_row": 2e-8,
     "materialize_ms_per_byte": 2e-10, "group_ms_per_key": 1e-8, "sync_ms": 0.012,
     "exec_overhead_ms": 0.02, "build_overhead_ms": 0.01, "dedup_overhead_ms": 0.01}


def shape(**kw):
    d = dict(n_r=1_000_000, n_s=1_000_000, n_rp=1_000_000, n_sp=1_000_000, n_distinct=250_000, sum_k=4_000_000,
             survivors=60_000, key_bytes=4, payload_bytes=4, sort_passes=3, dedup_passes=3, corr_op="=", agg="min")
    d.update(kw)
    return d


def test_best_is_argmin_and_all_strategies_present():
    for op in ("=", "<", "!="):
        for agg in ("min", "count", "sum", "avg", "exists"):
            e = cost_estimate(P, **shape(corr_op=op, agg=agg, payload_bytes=0 if agg in ("count", "exists") else 4))
            ms = {s: e[s] for s in STRATEGIES}
            assert all(v > 0 and math.isfinite(v) for v in ms.values())
            assert e["best"] == min(ms, key=ms.get)


def test_nested_part_scales_with_evaluations():
    """Eq. (6): N = (S - Ch) * per-evaluation cost + invariant parts."""
    a = cost_estimate(P, **shape(corr_op="<", n_rp=400_000, n_distinct=100_000, survivors=0))
    b = cost_estimate(P, **shape(corr_op="<", n_rp=800_000, n_distinct=100_000, survivors=0))
    # S' selection (one filter launch) + init + nested-loop launches
    inv = P["launch_ms"] + P["filter_ms_per_row"] * 1_000_000 + 2 * P["launch_ms"]
    na, nb = a["nested"]["nested_loop"] - inv, b["nested"]["nested_loop"] - inv
    assert nb == pytest.approx(2 * na, rel=1e-9)
    # caching evaluates each distinct value once: the pair term drops to n_distinct / n_rp of it
    pair_a = P["bnl_ms_per_pair"][0][0] * 400_000 * 1_000_000
    pair_c = P["bnl_ms_per_pair"][0][0] * 100_000 * 1_000_000
    assert a["nested"]["nested_loop"] - a["nested"]["nested_loop_cached"] > 0.9 * (pair_a - pair_c) - 1.0


def test_invariant_parts_do_not_depend_on_outer_size():
    a = cost_estimate(P, **shape(n_rp=1000, n_distinct=1000, sum_k=4000))
    b = cost_estimate(P, **shape(n_rp=900_000, n_distinct=200_000, sum_k=3_600_000))
    assert a["index_build_ms"] == b["index_build_ms"]


def test_launch_constant_is_per_launch_not_per_tuple():
    """Vectorisation: growing |R'| by 1000x adds only element costs."""
    small = cost_estimate(P, **shape(n_r=1000, n_rp=1000, n_distinct=1000, sum_k=4000, survivors=10))
    big = cost_estimate(P, **shape(n_r=1_000_000, n_rp=1_000_000, n_distinct=1_000_000, sum_k=4_000_000,
                                   survivors=10))
    per_tuple_c = (1_000_000 - 1000) * P["launch_ms"]   # what an unvectorised loop would add
    assert big["index"] - small["index"] < 0.01 * per_tuple_c


def test_index_wins_on_large_equality_and_loop_on_tiny_inputs():
    assert cost_estimate(P, **shape())["best"] in ("index", "index_cached")
    tiny = cost_estimate(P, **shape(n_r=4, n_s=64, n_rp=4, n_sp=64, n_distinct=4, sum_k=4, survivors=1,
                                    sort_passes=1, dedup_passes=1))
    assert tiny["nested_loop"] < tiny["index"]


@pytest.mark.parametrize("bad", [dict(n_rp=-1), dict(key_bytes=3), dict(payload_bytes=2), dict(sort_passes=9),
                                 dict(n_rp=2_000_000), dict(n_distinct=2_000_000)])
def test_rejects_bad_input(bad):
    with pytest.raises(NestGPUError):
        cost_estimate(P, **shape(**bad))


@pytest.mark.gpu
def test_calibrate_and_choose_on_gpu():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_icde_floratosxwgylz21_b200 import Engine
    eng = Engine(0, arena_bytes=2 << 30)
    try:
        p = eng.cost_calibrate(1 << 20).as_dict()
    finally:
        eng.close()
    flat = [v for k, v in p.items() if k != "bnl_ms_per_pair"] + p["bnl_ms_per_pair"][0] + p["bnl_ms_per_pair"][1]
    assert all(math.isfinite(v) and v >= 0 for v in flat)
    assert p["launch_ms"] > 0 and min(p["bnl_ms_per_pair"][0][:3]) > 0
    # integer-pipe bound: MIN pairs cost about 2x COUNT pairs;
    # 64-bit keys need a second compare
    assert p["bnl_ms_per_pair"][0][0] > 1.2 * p["bnl_ms_per_pair"][0][1]
    assert p["bnl_ms_per_pair"][1][1] > 1.2 * p["bnl_ms_per_pair"][0][1]
    assert cost_estimate(p, **shape())["best"] in ("index", "index_cached")


@pytest.mark.gpu
def test_exec_auto_matches_oracle_and_picks_index_for_large_equality():
    """nested.exec_auto runs the model's choice; the result is the oracle's
    whatever the choice (C1 small: nested loop; C2-shaped '=': index)."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import numpy as np
    import oracle
    from datagen import make_plan, query1
    from paper_conf_icde_floratosxwgylz21_b200 import Engine, nested
    eng = Engine(0, arena_bytes=2 << 30)
    try:
        params = eng.cost_calibrate(1 << 20)
        for t, want in ((query1.config("C1"), None), (query1.config("C2", n_r=50_000), "index")):
            plan = make_plan("=", "min", "=")
            n_r, n_s = len(t["R"]["col1"]), len(t["S"]["col1"])
            stats = dict(n_r=n_r, n_s=n_s, n_rp=n_r, n_sp=n_s, n_distinct=len(np.unique(t["R"]["col1"])),
                         sum_k=4 * n_r, survivors=n_r // 16, key_bytes=4, payload_bytes=4, sort_passes=3,
                         dedup_passes=3, corr_op="=", agg="min")
            m = eng.mark()
            R, S = eng.load_table(t["R"]), eng.load_table(t["S"])
            res, strategy, _ = nested.exec_auto(eng, plan, R, S, params, stats)
            g = eng.result_to_numpy(res)
            eng.release(m)
            rows, vals = oracle.survivors(oracle.evaluate(t, plan))
            assert np.array_equal(g["row"], rows) and np.array_equal(g["value"], vals), strategy
            if want:
                assert strategy.startswith(want), strategy
    finally:
        eng.close()


@pytest.mark.parametrize("bits,lo,kb,want", [
    (18, 0, 4, 2),    # C2 keys U[0, 2^18): two 9-bit passes instead of three 8-bit ones
    (21, 5, 4, 3),    # multiples of 32 below 2^26: windows at 5, 13, 21
    (26, 0, 4, 4),    # 4 x 8 bits (3 x 9 would not pay)
    (31, 0, 4, 4),
    (8, 0, 4, 1),
    (1, 7, 4, 1),
    (0, 0, 4, 0),     # all keys equal: nothing to sort
    (25, 20, 8, 4),   # 64-bit keys, bits 20..44 vary (windows cross bit 32)
    (64, 0, 8, 8),
])
def test_sort_pass_plan_mirror(bits, lo, kb, want):
    """tools/cost_model._passes mirrors the engine's radix-pass planner
    (api.cpp plan_sort_passes): greedy windows over the varying key bits,
    9-bit windows only when they need <= 2/3 of the 8-bit passes."""
    import numpy as np
    from tools.cost_model import _passes
    dt = np.uint32 if kb == 4 else np.uint64
    if bits == 0:
        keys = np.array([5, 5, 5], dtype=dt)
    else:
        top = (1 << bits) - 1
        keys = np.array([0, top << lo], dtype=np.uint64).astype(dt)
    assert _passes(keys, kb) == want


def test_stats_key_ordered_column_needs_no_sort():
    """tools/cost_model.stats mirrors the engine's key-ordered index build:
    a NOT NULL inner key column stored in ascending order (TPC-H lineitem by
    l_orderkey) has no sort passes; the same column shuffled, or with NULLs,
    keeps its radix passes."""
    import numpy as np
    from datagen import make_plan
    from tools.cost_model import stats
    rng = np.random.default_rng(1)
    k = np.sort(rng.integers(0, 1 << 24, 5000)).astype(np.int32)
    t = {"R": {"col1": k[:100].copy(), "col2": np.zeros(100, np.int32)},
         "S": {"col1": k, "col2": rng.integers(0, 9, 5000).astype(np.int32)}}
    plan = make_plan("=", "min", "=")
    assert stats(t, plan, 0)["sort_passes"] == 0
    t["S"]["col1"] = rng.permutation(k)
    assert stats(t, plan, 0)["sort_passes"] == 3
    t["S"]["col1"] = k
    t["S_valid"] = {"col1": np.ones(5000, bool)}
    assert stats(t, plan, 0)["sort_passes"] == 3
