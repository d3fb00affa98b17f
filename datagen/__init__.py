"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This package produces INPUTS ONLY (columns, NULL masks and plan descriptions).
It holds none of the method's arithmetic: no predicate evaluation, no aggregate,
no comparison of outer and inner tuples.  Both `oracle/` and the product
binding consume what it returns; neither imports the other.

Recipes (all numpy ``Generator(PCG64(seed))``):

* ``query1``  -- PAPER.md P:41 (Query 1) / P:53 (non-equality variant):
  R(col1, col2), S(col1, col2) int32.  Key / value ranges per config are
  listed in DESIGN.md "Input recipe" and in :data:`query1.CONFIGS`.
* ``tpch``    -- TPC-H-shaped base tables and their flattening into the plan
  template's R / S (PAPER.md P:227 join-first, P:319-329 invariant hoisting).
"""
from .plans import make_plan, PLAN_OPS, PLAN_AGGS  # noqa: F401
from . import query1  # noqa: F401
