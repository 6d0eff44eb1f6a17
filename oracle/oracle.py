"""Python wrapper of the CPU oracle (oracle/mdh_oracle.c).  TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg and --impl
reference) may import this module.  It shares no code with the CUDA path and does
not import it: it encodes the spec dict (mdh_workloads.specs) in the oracle's own
integer format and calls the C loop nest through ctypes.

Outputs: float buffers come back as float64 arrays (the fp64 oracle result, reading
C-13); integer buffers in their own dtype.  Elements outside the image of the output
index functions keep the caller's fill value (reading C-5).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "mdh_oracle.c")
LIB = os.path.join(HERE, "libmdh_oracle.so")

MAGIC = 0x4D44484F
_DT = {"bf16": 0, "f32": 1, "f64": 2, "i32": 3, "u32": 4, "i64": 5}
_OP = {"CC": 0, "PW_ADD": 1, "PW_MAX": 2, "PW_MIN": 3, "PW_PRL_ARGMAX": 4, "PW_PRL_PAPER": 5, "PS_ADD": 6}
_FN = {"MUL": 0, "STENCIL": 1, "PRL_COMPARE": 2, "IDENTITY": 3}
_NP_IN = {"bf16": np.uint16, "f32": np.float32, "f64": np.float64, "i32": np.int32,
          "u32": np.uint32, "i64": np.int64}
_NP_OUT = {"bf16": np.float64, "f32": np.float64, "f64": np.float64, "i32": np.int32,
           "u32": np.uint32, "i64": np.int64}
FLOAT = ("bf16", "f32", "f64")

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with -O2 -fno-fast-math -ffp-contract=off (no FMA contraction,
    reading C-13) and OpenMP.  The build of the checker is not a use of it."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        tmp = LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp",
                               "-std=c11", "-Wall", "-shared", "-fPIC", SRC, "-o", tmp])
        os.replace(tmp, LIB)
    return LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(LIB)
            P, I64, I = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
            L.mdho_shapes.argtypes = [P, I64, P, I, P, ctypes.c_char_p, I]
            L.mdho_eval.argtypes = [P, I64, P, I, P, P, I, ctypes.c_char_p, I]
            L.mdho_eval_points.argtypes = [P, I64, P, I, P, I64, P, P, P, P, I, ctypes.c_char_p, I]
            L.mdho_combine_tuple.argtypes = [I, I, I, P, P, P, P]
            L.mdho_max_threads.restype = I
            _lib = L
    return _lib


class OracleError(RuntimeError):
    pass


def encode(spec: dict) -> tuple[np.ndarray, np.ndarray]:
    e = [MAGIC, spec["D"]]
    e += list(spec["sizes"])
    e += [_OP[o] for o in spec["ops"]]
    e += [_FN[spec["f"]], len(spec["inputs"]), len(spec["outputs"])]
    for buf in list(spec["inputs"]) + list(spec["outputs"]):
        rank = len(buf["acc"][0]["offset"])
        e += [_DT[buf["dtype"]], rank]
        e += list(buf["shape"]) if buf.get("shape") else [0] * rank
        e += [len(buf["acc"])]
        for acc in buf["acc"]:
            assert len(acc["coeff"]) == rank and len(acc["offset"]) == rank
            for row in acc["coeff"]:
                assert len(row) == spec["D"]
                e += list(row)
            e += list(acc["offset"])
    fp = np.asarray(spec.get("fparams", []), np.float64)
    return np.asarray(e, np.int64), np.ascontiguousarray(fp)


def _ptrs(arrs):
    return (ctypes.c_void_p * max(1, len(arrs)))(*[a.ctypes.data for a in arrs])


def shapes(spec: dict) -> list[list[int]]:
    enc, fp = encode(spec)
    nb = len(spec["inputs"]) + len(spec["outputs"])
    out = np.zeros(nb * 8, np.int64)
    err = ctypes.create_string_buffer(512)
    rc = lib().mdho_shapes(enc.ctypes.data, len(enc), fp.ctypes.data, len(fp), out.ctypes.data, err, 512)
    if rc != 0:
        raise OracleError(err.value.decode())
    res = []
    for b, buf in enumerate(list(spec["inputs"]) + list(spec["outputs"])):
        rank = len(buf["acc"][0]["offset"])
        res.append([int(x) for x in out[b * 8:b * 8 + rank]])
    return res


def _check_inputs(spec, inputs):
    shp = shapes(spec)
    arrs = []
    for b, (buf, x) in enumerate(zip(spec["inputs"], inputs)):
        x = np.ascontiguousarray(x)
        want = _NP_IN[buf["dtype"]]
        if x.dtype != want:
            raise OracleError(f"input {b} dtype {x.dtype} != {np.dtype(want)}")
        if int(np.prod(shp[b])) != x.size:
            raise OracleError(f"input {b} has {x.size} elements, spec needs {shp[b]}")
        arrs.append(x)
    return shp, arrs


def evaluate(spec: dict, inputs: list[np.ndarray], threads: int = 0, fill=None) -> list[np.ndarray]:
    """Evaluate the whole md_hom literally.  Returns one array per output buffer."""
    shp, arrs = _check_inputs(spec, inputs)
    nin = len(spec["inputs"])
    outs = []
    for b, buf in enumerate(spec["outputs"]):
        dt = _NP_OUT[buf["dtype"]]
        o = np.zeros(shp[nin + b], dt)
        if fill is not None:
            o[...] = fill if buf["dtype"] in FLOAT else 0
        outs.append(o)
    enc, fp = encode(spec)
    err = ctypes.create_string_buffer(512)
    rc = lib().mdho_eval(enc.ctypes.data, len(enc), fp.ctypes.data, len(fp), _ptrs(arrs),
                         _ptrs(outs), threads, err, 512)
    if rc != 0:
        raise OracleError(err.value.decode())
    return outs


def evaluate_points(spec: dict, inputs: list[np.ndarray], points: np.ndarray, threads: int = 0):
    """Evaluate at sampled cc points (points: [n, D] int64, pw entries ignored).
    Returns (lin [n_out, n], values list per output buffer)."""
    _, arrs = _check_inputs(spec, inputs)
    pts = np.ascontiguousarray(points, np.int64)
    n = pts.shape[0]
    nout = len(spec["outputs"])
    lin = np.zeros((nout, n), np.int64)
    vf = np.zeros((nout, n), np.float64)
    vi = np.zeros((nout, n), np.int64)
    enc, fp = encode(spec)
    err = ctypes.create_string_buffer(512)
    rc = lib().mdho_eval_points(enc.ctypes.data, len(enc), fp.ctypes.data, len(fp), _ptrs(arrs), n,
                                pts.ctypes.data, lin.ctypes.data, vf.ctypes.data, vi.ctypes.data,
                                threads, err, 512)
    if rc != 0:
        raise OracleError(err.value.decode())
    vals = [vf[b] if spec["outputs"][b]["dtype"] in FLOAT else vi[b] for b in range(nout)]
    return lin, vals


def combine_tuple(op: str, f: str, kind: int, lhs, rhs):
    """⊕(lhs, rhs) for one tuple (f64[3], i64[3]) — exposes the oracle's catalog combine
    for the operator-algebra tests (kind: 0 float, 1 i32, 2 u32, 3 i64, 4 PRL)."""
    lf = np.ascontiguousarray(lhs[0], np.float64).copy()
    li = np.ascontiguousarray(lhs[1], np.int64).copy()
    rf = np.ascontiguousarray(rhs[0], np.float64)
    ri = np.ascontiguousarray(rhs[1], np.int64)
    lib().mdho_combine_tuple(_OP[op], _FN[f], kind, lf.ctypes.data, li.ctypes.data,
                             rf.ctypes.data, ri.ctypes.data)
    return lf, li


def max_threads() -> int:
    return int(lib().mdho_max_threads())


def random_points(spec: dict, n: int, seed: int = 7) -> np.ndarray:
    g = np.random.Generator(np.random.PCG64(seed))
    pts = np.zeros((n, spec["D"]), np.int64)
    for d, (s, o) in enumerate(zip(spec["sizes"], spec["ops"])):
        if o == "CC":
            pts[:, d] = g.integers(0, s, size=n)
    return pts


def stencil_sweeps(spec: dict, u0: np.ndarray, sweeps: int, threads: int = 0) -> np.ndarray:
    """`sweeps` applications of a same-shape all-cc map (reading C-34):
    u_{t+1} = md_hom(f, cc…)(u_t) on the image of the output index function, u_t elsewhere
    (the fixed boundary, reading C-5).  A plain loop over evaluate(); the state is kept in
    fp64 (the spec is re-typed to f64 after the first application).  Returns fp64."""
    if len(spec["inputs"]) != 1 or len(spec["outputs"]) != 1 or any(o != "CC" for o in spec["ops"]):
        raise OracleError("stencil_sweeps needs one input, one output and only cc dims")
    sp64 = {**spec, "inputs": [{**spec["inputs"][0], "dtype": "f64"}],
            "outputs": [{**spec["outputs"][0], "dtype": "f64"}]}
    u = np.ascontiguousarray(u0, np.float64).copy()
    for _ in range(sweeps):
        nxt = evaluate(sp64, [u], threads=threads, fill=np.nan)[0].reshape(u.shape)
        u = np.where(np.isnan(nxt), u, nxt)
    return u

