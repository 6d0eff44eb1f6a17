"""Thin ctypes binding of libmdh (include/mdh.h) — argument marshalling only.

Every step of the computation runs in libmdh's sm_100a kernels; PyTorch is used for
device memory, streams and process groups.  There is no CPU fallback: if the CUDA
library is missing, importing/using this module raises.

Spec dicts are the ones of ``mdh_workloads.specs`` (the paper's problem statement:
sizes, one combine operator per dimension, a catalog scalar function, affine index
functions for inputs and outputs; Listing 7, Listing 14).
"""
from __future__ import annotations

import ctypes
import json
import os
import threading

import numpy as np

MAX_D, MAX_RANK, MAX_ACC, MAX_BUFS = 10, 8, 32, 32
ABI_VERSION = 3                    # include/mdh.h MDH_ABI_VERSION
HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libmdh.so")

DTYPE = {"bf16": 0, "f32": 1, "f64": 2, "i32": 3, "u32": 4, "i64": 5}
DTYPE_NAME = {v: k for k, v in DTYPE.items()}
OP = {"CC": 0, "PW_ADD": 1, "PW_MAX": 2, "PW_MIN": 3, "PW_PRL_ARGMAX": 4, "PW_PRL_PAPER": 5, "PS_ADD": 6}
FN = {"MUL": 0, "STENCIL": 1, "PRL_COMPARE": 2, "IDENTITY": 3}
STATUS = {0: "OK", 1: "INVALID_ARG", 2: "INVALID_SPEC", 3: "UNSUPPORTED", 4: "OUT_OF_MEMORY",
          5: "CUDA", 6: "NCCL", 7: "INTERNAL"}
VIRTUAL_SHARD = 0x1
NO_COLLECTIVE = 0x2
FLOAT_ALLREDUCE = 0x4                # include/mdh.h MDH_PLAN_FLOAT_ALLREDUCE


class IndexFn(ctypes.Structure):
    _fields_ = [("coeff", (ctypes.c_int64 * MAX_D) * MAX_RANK), ("offset", ctypes.c_int64 * MAX_RANK)]


class Buffer(ctypes.Structure):
    _fields_ = [("dtype", ctypes.c_int), ("rank", ctypes.c_int32), ("shape", ctypes.c_int64 * MAX_RANK),
                ("n_acc", ctypes.c_int32), ("acc", IndexFn * MAX_ACC)]


class Spec(ctypes.Structure):
    _fields_ = [("D", ctypes.c_int32), ("size", ctypes.c_int64 * MAX_D), ("op", ctypes.c_int * MAX_D),
                ("f", ctypes.c_int), ("n_fparams", ctypes.c_int32), ("fparams", ctypes.POINTER(ctypes.c_double)),
                ("n_in", ctypes.c_int32), ("in_", ctypes.POINTER(Buffer)),
                ("n_out", ctypes.c_int32), ("out", ctypes.POINTER(Buffer))]


class PlanOpts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("world_size", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("nccl_comm", ctypes.c_void_p), ("shard_dim", ctypes.c_int32), ("flags", ctypes.c_uint32),
                ("tile_table", ctypes.c_char_p), ("force_tile", ctypes.c_char_p)]


class Halo(ctypes.Structure):
    """mdh_halo (include/mdh.h): the z-slab neighbourhood of a stencil time-stepping rank."""
    _fields_ = [("nccl_comm", ctypes.c_void_p), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("peer_lo", ctypes.c_void_p * 2), ("peer_hi", ctypes.c_void_p * 2)]


class MdhError(RuntimeError):
    def __init__(self, status, msg):
        self.status = STATUS.get(status, str(status))
        super().__init__(f"mdh {self.status}: {msg}")


_lib = None
_lock = threading.Lock()


def library_path() -> str:
    return LIB_PATH


def lib():
    """Load libmdh.so (built by paper_conf_sc_schulzegr25_b200.build); raises if absent."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise ImportError(f"{LIB_PATH} is missing: build it with "
                                  "`python -m paper_conf_sc_schulzegr25_b200.build` (there is no CPU fallback)")
            L = ctypes.CDLL(LIB_PATH)
            P, S = ctypes.c_void_p, ctypes.c_size_t
            L.mdh_plan.argtypes = [ctypes.POINTER(Spec), ctypes.POINTER(PlanOpts), ctypes.POINTER(P)]
            L.mdh_plan_workspace_size.argtypes = [P, ctypes.POINTER(S)]
            L.mdh_plan_local_shape.argtypes = [P, ctypes.c_int32, ctypes.c_int32, P, P, P, P]
            L.mdh_plan_describe.argtypes = [P, ctypes.c_char_p, S, ctypes.POINTER(S)]
            L.mdh_execute.argtypes = [P, P, P, P, S, P]
            L.mdh_plan_host_scratch_size.argtypes = [P, ctypes.POINTER(S)]
            L.mdh_execute_host.argtypes = [P, P, P, P, S, P]
            L.mdh_combine_partials.argtypes = [P, P, ctypes.c_int32, P, P]
            L.mdh_destroy.argtypes = [P]
            L.mdh_comm_unique_id.argtypes = [P]
            L.mdh_comm_init.argtypes = [P, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.POINTER(P)]
            L.mdh_comm_destroy.argtypes = [P]
            L.mdh_last_error.restype = ctypes.c_char_p
            L.mdh_abi_version.restype = ctypes.c_int32
            L.mdh_last_launch_count.restype = ctypes.c_int32
            L.mdh_stencil_sweeps.argtypes = [P, P, P, ctypes.c_int32, ctypes.POINTER(Halo), P, S, P,
                                             ctypes.POINTER(ctypes.c_int32)]
            D = ctypes.POINTER(ctypes.c_double)
            L.mdh_measure_peaks.argtypes = [ctypes.c_int32, D, D, D]
            L.mdh_measure_peaks.restype = ctypes.c_int
            L.mdh_debug_t4_trace.argtypes = [P, ctypes.c_int64]
            L.mdh_debug_t4_trace.restype = ctypes.c_int64
            for name in ("mdh_plan", "mdh_plan_workspace_size", "mdh_plan_local_shape", "mdh_plan_describe",
                         "mdh_execute", "mdh_plan_host_scratch_size", "mdh_execute_host",
                         "mdh_combine_partials", "mdh_destroy", "mdh_comm_unique_id", "mdh_comm_init",
                         "mdh_comm_destroy", "mdh_stencil_sweeps"):
                getattr(L, name).restype = ctypes.c_int
            if L.mdh_abi_version() != ABI_VERSION:
                raise RuntimeError(f"{LIB_PATH}: ABI version {L.mdh_abi_version()} != {ABI_VERSION} (stale build?)")
            _lib = L
    return _lib


def _check(status):
    if status != 0:
        raise MdhError(status, lib().mdh_last_error().decode(errors="replace"))


def _fill_buffer(cb: Buffer, buf: dict, D: int):
    cb.dtype = DTYPE[buf["dtype"]]
    rank = len(buf["acc"][0]["offset"])
    cb.rank = rank
    shape = buf.get("shape") or [0] * rank
    for r in range(rank):
        cb.shape[r] = int(shape[r])
    cb.n_acc = len(buf["acc"])
    for a, acc in enumerate(buf["acc"]):
        for r in range(rank):
            cb.acc[a].offset[r] = int(acc["offset"][r])
            for d in range(D):
                cb.acc[a].coeff[r][d] = int(acc["coeff"][r][d])


def make_cspec(spec: dict):
    """Marshal a spec dict into the C structs (kept alive by the returned tuple)."""
    s = Spec()
    s.D = spec["D"]
    for d in range(spec["D"]):
        s.size[d] = int(spec["sizes"][d])
        s.op[d] = OP[spec["ops"][d]]
    s.f = FN[spec["f"]]
    fp = (ctypes.c_double * max(1, len(spec.get("fparams", []))))(*spec.get("fparams", []))
    s.n_fparams = len(spec.get("fparams", []))
    s.fparams = ctypes.cast(fp, ctypes.POINTER(ctypes.c_double))
    ins = (Buffer * len(spec["inputs"]))()
    outs = (Buffer * len(spec["outputs"]))()
    for b, buf in enumerate(spec["inputs"]):
        _fill_buffer(ins[b], buf, spec["D"])
    for b, buf in enumerate(spec["outputs"]):
        _fill_buffer(outs[b], buf, spec["D"])
    s.n_in, s.in_ = len(spec["inputs"]), ctypes.cast(ins, ctypes.POINTER(Buffer))
    s.n_out, s.out = len(spec["outputs"]), ctypes.cast(outs, ctypes.POINTER(Buffer))
    return s, (fp, ins, outs)


def torch_dtype(name):
    import torch
    return {"bf16": torch.bfloat16, "f32": torch.float32, "f64": torch.float64, "i32": torch.int32,
            "u32": torch.uint32, "i64": torch.int64}[name]


def to_device(x: np.ndarray, dtype: str, device):
    """numpy host array (bf16 given as uint16 bit patterns) → torch tensor on `device`."""
    import torch
    if dtype == "bf16":
        t = torch.from_numpy(np.ascontiguousarray(x).view(np.int16)).view(torch.bfloat16)
    elif dtype == "u32":
        t = torch.from_numpy(np.ascontiguousarray(x).view(np.int32)).view(torch.uint32)
    else:
        t = torch.from_numpy(np.ascontiguousarray(x))
    return t.to(device)


def to_numpy(t, dtype: str) -> np.ndarray:
    import torch
    t = t.detach().cpu().contiguous()
    if dtype == "bf16":
        return t.view(torch.int16).numpy().view(np.uint16)
    if dtype == "u32":
        return t.view(torch.int32).numpy().view(np.uint32)
    return t.numpy()


class Plan:
    """A planned MDH computation (mdh_plan).  Call it with device tensors."""

    def __init__(self, spec: dict, device=None, world_size=1, rank=0, comm=None, shard_dim=-1, flags=0,
                 tile_table=None, force_tile=None):
        self.spec = spec
        cs, self._keep = make_cspec(spec)
        o = PlanOpts()
        if device is None:
            device = 0
        self.device_index = int(getattr(device, "index", device) or 0)
        o.device = self.device_index
        o.world_size, o.rank = int(world_size), int(rank)
        o.nccl_comm = comm.handle if isinstance(comm, Comm) else comm
        o.shard_dim, o.flags = int(shard_dim), int(flags)
        o.tile_table = tile_table.encode() if tile_table else None
        o.force_tile = force_tile.encode() if force_tile else None
        h = ctypes.c_void_p()
        _check(lib().mdh_plan(ctypes.byref(cs), ctypes.byref(o), ctypes.byref(h)))
        self._h = h
        n = ctypes.c_size_t()
        _check(lib().mdh_plan_workspace_size(h, ctypes.byref(n)))
        self.workspace_bytes = n.value
        self.in_shapes = [self.local_shape(False, b)[0] for b in range(len(spec["inputs"]))]
        self.out_shapes = [self.local_shape(True, b)[0] for b in range(len(spec["outputs"]))]
        self._ws = None

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value:
            try:
                lib().mdh_destroy(h)
            except Exception:
                pass
            self._h = None

    def local_shape(self, is_output: bool, b: int):
        shp = (ctypes.c_int64 * MAX_RANK)()
        off = (ctypes.c_int64 * MAX_RANK)()
        dt = ctypes.c_int32()
        rk = ctypes.c_int32()
        _check(lib().mdh_plan_local_shape(self._h, int(is_output), b, shp, off, ctypes.byref(dt), ctypes.byref(rk)))
        return [shp[r] for r in range(rk.value)], [off[r] for r in range(rk.value)], DTYPE_NAME[dt.value]

    def describe(self) -> dict:
        need = ctypes.c_size_t()
        lib().mdh_plan_describe(self._h, None, 0, ctypes.byref(need))
        buf = ctypes.create_string_buffer(need.value)
        _check(lib().mdh_plan_describe(self._h, buf, need.value, None))
        return json.loads(buf.value.decode())

    @property
    def template(self) -> str:
        return self.describe()["template"]

    def empty_outputs(self, device=None):
        import torch
        dev = device if device is not None else torch.device("cuda", self.device_index)
        return [torch.empty(s, dtype=torch_dtype(b["dtype"]), device=dev)
                for s, b in zip(self.out_shapes, self.spec["outputs"])]

    def workspace(self, device=None):
        import torch
        if self._ws is None or self._ws.numel() < self.workspace_bytes + 256:
            dev = device if device is not None else torch.device("cuda", self.device_index)
            # zero-filled once (mdh.h workspace contract); executes keep it consistent
            self._ws = torch.zeros(self.workspace_bytes + 256, dtype=torch.uint8, device=dev)
        p = self._ws.data_ptr()
        return (p + 255) // 256 * 256

    def __call__(self, inputs, outputs=None, stream=None, workspace_ptr=None):
        import torch
        if outputs is None:
            outputs = self.empty_outputs(inputs[0].device)
        ip = (ctypes.c_void_p * len(inputs))(*[t.data_ptr() for t in inputs])
        op = (ctypes.c_void_p * len(outputs))(*[t.data_ptr() for t in outputs])
        ws = workspace_ptr if workspace_ptr is not None else (self.workspace() if self.workspace_bytes else None)
        st = stream if stream is not None else torch.cuda.current_stream(inputs[0].device).cuda_stream
        _check(lib().mdh_execute(self._h, ip, op, ws, self.workspace_bytes, st))
        return outputs

    def host_scratch_bytes(self) -> int:
        n = ctypes.c_size_t()
        _check(lib().mdh_plan_host_scratch_size(self._h, ctypes.byref(n)))
        return n.value

    def execute_host(self, host_inputs, host_outputs, scratch_ptr: int, scratch_bytes: int, stream: int):
        """End-to-end call: host (pinned) tensors in/out, copies inside (mdh_execute_host)."""
        ip = (ctypes.c_void_p * len(host_inputs))(*[t.data_ptr() for t in host_inputs])
        op = (ctypes.c_void_p * len(host_outputs))(*[t.data_ptr() for t in host_outputs])
        _check(lib().mdh_execute_host(self._h, ip, op, scratch_ptr, scratch_bytes, stream))

    def combine_partials(self, partials, outputs=None, stream=None):
        """Ordered ⊗-fold of S partial output sets (partials[s][b] device tensors)."""
        import torch
        if outputs is None:
            outputs = self.empty_outputs(partials[0][0].device)
        flat = [t for ps in partials for t in ps]
        pp = (ctypes.c_void_p * len(flat))(*[t.data_ptr() for t in flat])
        op = (ctypes.c_void_p * len(outputs))(*[t.data_ptr() for t in outputs])
        st = stream if stream is not None else torch.cuda.current_stream(outputs[0].device).cuda_stream
        _check(lib().mdh_combine_partials(self._h, pp, len(partials), op, st))
        return outputs

    def stencil_sweeps(self, u, v, sweeps: int, halo: "Halo | None" = None, stream=None, workspace_ptr=None):
        """Time-stepping (mdh_stencil_sweeps): `sweeps` applications u→v→u…, with the halo
        exchange of `halo` after each; returns the tensor holding the final field."""
        import torch
        ws = workspace_ptr if workspace_ptr is not None else (self.workspace() if self.workspace_bytes else None)
        st = stream if stream is not None else torch.cuda.current_stream(u.device).cuda_stream
        res = ctypes.c_int32()
        _check(lib().mdh_stencil_sweeps(self._h, u.data_ptr(), v.data_ptr(), sweeps,
                                        ctypes.byref(halo) if halo is not None else None, ws, self.workspace_bytes,
                                        st, ctypes.byref(res)))
        return v if res.value else u

    @staticmethod
    def last_launch_count() -> int:
        return int(lib().mdh_last_launch_count())

    @staticmethod
    def t4_trace(max_units: int = 65536):
        """Diagnostics: the T4 2-SM per-unit timeline of the last launch (MDH_T4_TRACE=1),
        as a list of (sm, pair, t_first_mma, t_last_commit, t_epilogue_done) in ns and
        (wait_full, wait_accumulator) in SM cycles, then (t_partials_seen, t_partial_published)
        in ns (stream-K finisher / producer units, else 0); and per CTA its (entry, exit) times."""
        buf = (ctypes.c_uint64 * (8 * max_units + 1024))()
        n = int(lib().mdh_debug_t4_trace(buf, max_units))
        if n < 0:
            raise MdhError(-1, "mdh_debug_t4_trace failed")
        units = [(buf[8 * u] >> 32, buf[8 * u] & 0xffffffff, buf[8 * u + 1], buf[8 * u + 2], buf[8 * u + 3],
                  buf[8 * u + 4], buf[8 * u + 5], buf[8 * u + 6], buf[8 * u + 7]) for u in range(n) if buf[8 * u + 1]]
        ee = [(buf[8 * n + i], buf[8 * n + i + 1]) for r in (0, 512) for i in range(r, r + 512, 2) if buf[8 * n + i]]
        return units, ee


class Comm:
    """NCCL communicator created through libmdh, bootstrapped over torch.distributed."""

    def __init__(self, group=None, device=None):
        import torch
        import torch.distributed as dist
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        idbuf = (ctypes.c_uint8 * 128)()
        if self.rank == 0:
            _check(lib().mdh_comm_unique_id(idbuf))
        backend = dist.get_backend(group)
        dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
        t = torch.tensor(list(bytes(idbuf)), dtype=torch.uint8,
                         device=dev if backend == "nccl" else "cpu")
        dist.broadcast(t, src=0, group=group)
        raw = bytes(t.cpu().tolist())
        ctypes.memmove(idbuf, raw, 128)
        h = ctypes.c_void_p()
        _check(lib().mdh_comm_init(idbuf, self.world, self.rank, int(dev.index or 0), ctypes.byref(h)))
        self.handle = h.value

    def close(self):
        if self.handle:
            lib().mdh_comm_destroy(self.handle)
            self.handle = None


def measure_peaks(device: int = 0) -> dict:
    """Measured FFMA / ALU-pipe / issue throughput of `device` (mdh_measure_peaks)."""
    f, a, i = ctypes.c_double(), ctypes.c_double(), ctypes.c_double()
    _check(lib().mdh_measure_peaks(int(device), ctypes.byref(f), ctypes.byref(a), ctypes.byref(i)))
    return {"ffma_tflops": f.value, "alu_tops": a.value, "issue_tops": i.value}


def abi_version() -> int:
    return int(lib().mdh_abi_version())
