"""CPU oracle for the nested-method correlated subquery.

TEST INFRASTRUCTURE ONLY -- see nestgpu_oracle.c's header.  Importable by
tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference legs.
"""
from .oracle import evaluate, collect, in_list, survivors, build, max_threads, OracleOverflow  # noqa: F401
