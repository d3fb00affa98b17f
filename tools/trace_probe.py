"""Host-side trace (NESTGPU_TRACE=1) of small queries: per-step host time of
build_index / exec, last of 30 runs per case (stderr)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["NESTGPU_TRACE"] = "1"


def main():
    import torch
    from datagen import make_plan, query1, tpch
    from paper_conf_icde_floratosxwgylz21_b200 import Engine
    from tests.gpu_helpers import load
    eng = Engine(0, arena_bytes=2 << 30)
    q2, p2 = tpch.flattened("q2", 1.0, 3)
    for name, t, plan, use_index in (("C1 > min", query1.config("C1"), make_plan(">", "min", "="), False),
                                     ("C1 = min", query1.config("C1"), make_plan("=", "min", "="), True),
                                     ("SF1 Q2", q2, p2, True)):
        m0 = eng.mark()
        R, S = load(eng, t)
        for i in range(30):
            if i >= 27:
                sys.stderr.write("--- %s\n" % name)
                sys.stderr.flush()
            m = eng.mark()
            idx = eng.index_for_plan(plan, S) if use_index else -1
            eng.exec(plan, R, S, index=idx)
            eng.release(m)
            torch.cuda.synchronize()
            sys.stderr.flush()
        eng.release(m0)


if __name__ == "__main__":
    main()
