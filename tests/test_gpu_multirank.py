"""The multi-GPU path end to end on one B200: two ranks (torch.distributed,
gloo, both processes on cuda:0 -- the box this suite runs on has one GPU)
shard R, receive S and the index by broadcast from rank 0, run both subquery
kernels on their shard, and gather the survivors to rank 0, which compares
them with the oracle on the whole of R (outer tuples are independent,
P:127-131).  The NCCL version of the same code runs under torchrun."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from datagen import make_plan, query1
        from paper_conf_icde_floratosxwgylz21_b200 import Engine, dist as ngd
        t = query1.tables(n_r=30011, n_s=20021, key_hi=4000, val_hi=16, seed=21)
        n_r, n_s = len(t["R"]["col1"]), len(t["S"]["col1"])
        lo, hi = ngd.shard_range(n_r, rank, world)
        eng = Engine(0, arena_bytes=256 << 20)
        R = eng.load_table({k: v[lo:hi] for k, v in t["R"].items()})
        S = ngd.share_table(eng, t["S"] if rank == 0 else None, ["col1", "col2"], n_s)
        ok = True
        for op, agg, mode in (("=", "min", "index"), ("=", "count", "index"), (">", "min", "bnl"),
                              ("!=", "count", "bnl"), ("<", "exists", "bnl"), ("=", "avg", "index")):
            plan = make_plan(op, agg, "<=")
            idx = ngd.share_index(eng, S, ["col1"], "col2" if agg in ("min", "avg") else None) if mode == "index" else -1
            res = eng.exec(plan, R, S, index=idx, row_id_base=lo)
            g = ngd.gather_result(eng, res)
            if rank == 0:
                ref = oracle.evaluate(t, plan)
                er, ev = oracle.survivors(ref)
                ok = ok and np.array_equal(g[0].cpu().numpy(), er) and np.array_equal(g[1].cpu().numpy(), ev)
        if rank == 0:
            q.put(("ok", ok))
        eng.close()
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e)))
        raise
    finally:
        dist.destroy_process_group()


def test_two_ranks_share_index_and_gather():
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(300)
    assert all(p.exitcode == 0 for p in ps)
    status, ok = q.get(timeout=10)
    assert status == "ok" and ok is True


def _peer_worker(rank, world, port, q, index_mode):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from datagen import make_plan, query1
        from paper_conf_icde_floratosxwgylz21_b200 import Engine, dist as ngd
        t = query1.tables(n_r=40009, n_s=20011, key_hi=3000, val_hi=16, seed=23)
        n_r, n_s = len(t["R"]["col1"]), len(t["S"]["col1"])
        lo, hi = ngd.shard_range(n_r, rank, world)
        eng = Engine(0, arena_bytes=256 << 20)
        R = eng.load_table({k: v[lo:hi] for k, v in t["R"].items()})
        S = ngd.share_table(eng, t["S"] if rank == 0 else None, ["col1", "col2"], n_s)
        pg = ngd.PeerGather(eng, n_r)
        ok, plans = True, 0
        for op, agg, mode in (("=", "min", "index"), ("<", "count", "bnl"), (">", "max", "bnl"),
                              ("!=", "exists", "bnl"), ("<=", "sum", "index"), ("=", "avg", "index")):
            plan = make_plan(op, agg, ">")
            payload = "col2" if agg in ("min", "max", "sum", "avg") else None
            idx = -1
            if mode == "index":
                idx = (eng.build_index(S, ["col1"], payload) if index_mode == "local"
                       else ngd.share_index(eng, S, ["col1"], payload))
            for rep in range(2):   # the window is reused across gathers
                res = eng.exec(plan, R, S, index=idx, row_id_base=lo)
                g = pg.gather(res)
                if rank == 0:
                    er, ev = oracle.survivors(oracle.evaluate(t, plan))
                    ok = ok and np.array_equal(g[0].cpu().numpy(), er) and np.array_equal(g[1].cpu().numpy(), ev)
                    plans += 1
        pg.close()
        if rank == 0:
            q.put(("ok", ok, plans))
        eng.close()
    except Exception as e:  # pragma: no cover
        q.put(("err", repr(e), 0))
        raise
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("index_mode", ["local", "broadcast"])
def test_two_ranks_peer_window_gather(index_mode):
    """The multi-GPU gather by peer stores: rank 0 creates a window
    (nestgpu_window_create, CUDA IPC), rank 1 maps it (nestgpu_window_open)
    and both store their survivors into it at their row offsets
    (nestgpu_result_put) from their own kernels; rank 0's window equals the
    oracle's whole-R survivors for both subquery kernels, with the index
    built on every rank or built on rank 0 and broadcast."""
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_peer_worker, args=(r, 2, port, q, index_mode)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(300)
    assert all(p.exitcode == 0 for p in ps)
    status, ok, plans = q.get(timeout=10)
    assert status == "ok" and ok is True and plans == 12
