"""Workload specs and seeded input generators shared by the oracle and the GPU path.

This package deliberately contains none of the method's arithmetic (no folds, no
combine operators, no scalar functions): see oracle/ for the CPU reference and
paper_conf_sc_schulzegr25_b200/ for the CUDA path.
"""
from . import specs, gen  # noqa: F401
