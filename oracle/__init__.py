"""CPU oracle of the MDH hot path — TEST INFRASTRUCTURE ONLY.

May be imported only by tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg,
--impl reference).  The product path (paper_conf_sc_schulzegr25_b200) never imports it.

Parity status of every oracle function is listed in DESIGN.md §3; all functions are
pinned by tests/test_oracle_*.py (closed forms, library routines, brute force,
homomorphism invariant, operator algebra).  No function is "parity unpinned" w.r.t.
the mathematics; parity with the AUTHORS' code is unpinned for the readings C-16,
C-18, C-19, C-21, C-22 because the paper prints no computed values.
"""
from .oracle import (evaluate, evaluate_points, shapes, combine_tuple, build,  # noqa: F401
                     max_threads, random_points, stencil_sweeps, OracleError)
