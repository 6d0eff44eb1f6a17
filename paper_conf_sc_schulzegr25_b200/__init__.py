"""B200-native (sm_100a) hot path of the MDH directive (Schulze, Gorlatch, Rasch, SC-W '25).

Evaluates md_hom(f, ⊗_1..⊗_D) over a D-dimensional index space behind the C-ABI of
include/mdh.h (libmdh.so, built from csrc/ by ``python -m paper_conf_sc_schulzegr25_b200.build``).
"""
from .mdh import (Plan, Comm, Halo, MdhError, lib, library_path, to_device, to_numpy, torch_dtype,  # noqa: F401
                  abi_version, measure_peaks, VIRTUAL_SHARD, NO_COLLECTIVE, FLOAT_ALLREDUCE)
