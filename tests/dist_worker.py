"""Worker for tests/test_dist_gloo.py::test_launch_ranks_world4: started by
paper_conf_icde_floratosxwgylz21_b200.dist.launch_ranks (torchrun, the path
bench.py --gpus N takes outside torchrun) with gloo on CPU.  Shards ONE R
(strong scaling, as bench.py does), evaluates each shard (the oracle stands
in for the engine: this covers the host plumbing, not the kernels), gathers
the survivors to rank 0 by point-to-point sends and compares them with the
whole-R evaluation.  Rank 0 writes its verdict to argv[1]."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402


def main(out_path):
    import oracle
    from datagen import make_plan, query1
    from paper_conf_icde_floratosxwgylz21_b200 import dist as ngd
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    t = query1.config("C1")
    n = len(t["R"]["col1"])
    verdict = {"world": world, "ok": True, "plans": 0}
    for op, agg in (("=", "min"), (">", "min"), ("!=", "count"), ("<", "exists")):
        plan = make_plan(op, agg, "=")
        lo, hi = ngd.shard_range(n, rank, world)
        if rank == world - 1:
            lo = hi  # the last rank holds an empty shard: zero-length sends must be skipped
        shard = {"R": {k: v[lo:hi] for k, v in t["R"].items()}, "S": t["S"]}
        res = oracle.evaluate(shard, plan)
        rows, vals = oracle.survivors(res)
        got = ngd.gather_rows([torch.from_numpy(rows + lo), torch.from_numpy(vals)])
        if rank == 0:
            R_cut = {k: v[:ngd.shard_range(n, world - 1, world)[0]] for k, v in t["R"].items()}
            er, ev = oracle.survivors(oracle.evaluate({"R": R_cut, "S": t["S"]}, plan))
            verdict["ok"] &= bool(np.array_equal(got[0].numpy(), er) and np.array_equal(got[1].numpy(), ev))
            verdict["plans"] += 1
        else:
            verdict["ok"] &= got is None
    counts = ngd.all_counts(rank + 1)
    verdict["counts_ok"] = counts == list(range(1, world + 1))
    verdict["max"] = ngd.max_over_ranks(float(rank))
    verdict["sum"] = ngd.sum_over_ranks(1.0)
    if rank == 0:
        with open(out_path, "w") as f:
            json.dump(verdict, f)
    dist.destroy_process_group()


if __name__ == "__main__":
    main(sys.argv[1])
