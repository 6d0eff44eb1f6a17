"""Seeded synthetic input generators (SURVEY §8(d).1 protocol; DESIGN.md §4 recipe).

Shared by the oracle tests and the GPU path.  Holds none of the method's arithmetic:
it only draws numbers (numpy PCG64, seed = 1000·config + buffer ordinal) shaped like
the paper's workloads (Fig 3).

bf16 inputs are represented as their raw 16-bit patterns (uint16 arrays), obtained by
round-to-nearest-even from the fp32 draws (reading C-15) — the same rounding as
``torch.Tensor.to(torch.bfloat16)``.  Both sides consume those exact bit patterns.
"""
from __future__ import annotations

import numpy as np

from . import specs as S

NP_DTYPE = {"bf16": np.uint16, "f32": np.float32, "f64": np.float64,
            "i32": np.int32, "u32": np.uint32, "i64": np.int64}


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(seed))


def f32_to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """Round fp32 → bf16 to nearest even; returns uint16 bit patterns (no NaNs drawn)."""
    u = np.ascontiguousarray(x, dtype=np.float32).view(np.uint32).astype(np.uint64)
    u = (u + 0x7FFF + ((u >> 16) & 1)) >> 16
    return u.astype(np.uint16)


def bf16_bits_to_f32(b: np.ndarray) -> np.ndarray:
    return (np.ascontiguousarray(b, dtype=np.uint16).astype(np.uint32) << 16).view(np.float32)


def buffer_shape(buf: dict, spec: dict) -> list[int]:
    """Declared shape, else the extent of the accessed index range (fn.7 P:316, C-9).
    Needed only to size host arrays; each side re-derives and validates it itself."""
    if buf.get("shape"):
        return list(buf["shape"])
    sizes = spec["sizes"]
    is_out = any(buf is o for o in spec["outputs"])
    rank = len(buf["acc"][0]["offset"])
    mx = [0] * rank
    for acc in buf["acc"]:
        for r in range(rank):
            hi = acc["offset"][r]
            for d, c in enumerate(acc["coeff"][r]):
                ext = sizes[d] - 1
                if is_out and spec["ops"][d] != "CC":
                    ext = 0
                hi += max(0, c * ext)
            mx[r] = max(mx[r], hi)
    return [m + 1 for m in mx]


def uniform(g, shape, lo, hi, dtype):
    x = g.uniform(lo, hi, size=shape).astype(np.float32)
    if dtype == "bf16":
        return f32_to_bf16_bits(x)
    return x.astype(NP_DTYPE[dtype])


def gen_inputs(spec: dict, seed_base: int, kind: str = "signed") -> list[np.ndarray]:
    """Generic generator: one array per input buffer, by dtype.
    kind: 'signed' (U[-1,1)), 'positive' (U[0.5,1.5)), 'ones', 'small_int'."""
    out = []
    for b, buf in enumerate(spec["inputs"]):
        shp = buffer_shape(buf, spec)
        g = rng(seed_base + b + 1)
        dt = buf["dtype"]
        if dt in ("f32", "f64", "bf16"):
            if kind == "positive":
                x = uniform(g, shp, 0.5, 1.5, dt)
            elif kind == "ones":
                x = np.ones(shp, np.float32)
                x = f32_to_bf16_bits(x) if dt == "bf16" else x.astype(NP_DTYPE[dt])
            else:
                x = uniform(g, shp, -1.0, 1.0, dt)
        elif dt in ("i32",):
            x = g.integers(-2 ** 15, 2 ** 15, size=shp, dtype=np.int64).astype(np.int32)
        elif dt == "u32":
            x = g.integers(0, 2 ** 32, size=shp, dtype=np.uint64).astype(np.uint32)
        else:
            x = g.integers(-2 ** 40, 2 ** 40, size=shp, dtype=np.int64)
        out.append(np.ascontiguousarray(x))
    return out


# ---------------------------------------------------------------------------------------
# Config-specific recipes (SURVEY §8(d).2 D-1 … D-5)
# ---------------------------------------------------------------------------------------

def dot_inputs(N, dtype="f32", kind="signed", seed_base=1000):
    g1, g2 = rng(seed_base + 1), rng(seed_base + 2)
    if dtype == "i32":
        if kind == "iota_one":       # closed form a_i = i, b_i = 1
            return [np.arange(N, dtype=np.int64).astype(np.uint32).view(np.int32), np.ones(N, np.int32)]
        if kind == "iota_iota":      # closed form a_i = b_i = i
            a = np.arange(N, dtype=np.int64).astype(np.uint32).view(np.int32)
            return [a, a.copy()]
        return [g1.integers(-2 ** 15, 2 ** 15, size=N, dtype=np.int64).astype(np.int32),
                g2.integers(-2 ** 15, 2 ** 15, size=N, dtype=np.int64).astype(np.int32)]
    lo, hi = (0.5, 1.5) if kind == "positive" else (-1.0, 1.0)
    return [uniform(g1, [N], lo, hi, dtype), uniform(g2, [N], lo, hi, dtype)]


def matmul_inputs(M, N, K, dtype="f32", kind="signed", seed_base=2000):
    g1, g2 = rng(seed_base + 1), rng(seed_base + 2)
    if kind == "ones":
        a = np.ones((M, K), np.float32)
        b = np.ones((K, N), np.float32)
    elif kind == "identity":
        assert M == K
        a = np.eye(M, dtype=np.float32)
        b = g2.uniform(-1, 1, size=(K, N)).astype(np.float32)
    else:
        lo, hi = (0.5, 1.5) if kind == "positive" else (-1.0, 1.0)
        a = g1.uniform(lo, hi, size=(M, K)).astype(np.float32)
        b = g2.uniform(lo, hi, size=(K, N)).astype(np.float32)
    if dtype == "bf16":
        return [f32_to_bf16_bits(a), f32_to_bf16_bits(b)]
    return [a, b]


def jacobi3d_inputs(Z, Y, X, kind="random", seed_base=3000):
    g = rng(seed_base + 1)
    if kind == "constant":
        return [np.full((Z, Y, X), 2.0, np.float32)]
    if kind == "linear":       # u = x + 2y + 3z (exact in fp32 for these sizes)
        z, y, x = np.indices((Z, Y, X), dtype=np.float32)
        return [np.ascontiguousarray(x + 2 * y + 3 * z, dtype=np.float32)]
    return [g.uniform(0.0, 1.0, size=(Z, Y, X)).astype(np.float32)]


def gaussian2d_inputs(I, J, kind="random", seed_base=3100):
    """Gaussian_2D image (I+4)×(J+4) fp32: U[0,1) pixel intensities, or closed-form fields."""
    if kind == "constant":
        return [np.full((I + 4, J + 4), 3.0, np.float32)]
    if kind == "linear":       # x + 2y (exact in fp32 for these sizes)
        y, x = np.indices((I + 4, J + 4), dtype=np.float32)
        return [np.ascontiguousarray(x + 2 * y, dtype=np.float32)]
    return [rng(seed_base + 1).uniform(0.0, 1.0, size=(I + 4, J + 4)).astype(np.float32)]


def ccsd_inputs(spec, kind="signed", seed_base=4000):
    return gen_inputs(spec, seed_base, kind)


def mcc_inputs(spec, seed_base=4100):
    """img: post-ReLU activations U[0,1) in the interior with a zero border (the
    enlarged buffer of P:312, fn. P:407-409); flt: He-normal N(0, sqrt(2/(R*S*C)))."""
    N, P, Q, K, R, Sx, C = spec["sizes"]
    ib, fb = spec["inputs"]
    H, W = ib["shape"][1], ib["shape"][2]
    g1, g2 = rng(seed_base + 1), rng(seed_base + 2)
    pad_h = (R - 1) // 2 if R > 1 else 0
    pad_w = (Sx - 1) // 2 if Sx > 1 else 0
    img = np.zeros((N, H, W, C), np.float32)
    ih, iw = H - 2 * pad_h, W - 2 * pad_w
    img[:, pad_h:pad_h + ih, pad_w:pad_w + iw, :] = g1.uniform(0.0, 1.0, size=(N, ih, iw, C))
    flt = g2.normal(0.0, np.sqrt(2.0 / (R * Sx * C)), size=(K, R, Sx, C)).astype(np.float32)
    if ib["dtype"] == "bf16":
        return [f32_to_bf16_bits(img), f32_to_bf16_bits(flt)]
    return [img, flt.astype(np.float32)]


def _zipf_codes(g, n, dom, a=1.1):
    z = g.zipf(a, size=n).astype(np.int64)
    return ((z - 1) % dom).astype(np.uint32)


def prl_inputs(N, I, seed_base=5000, dup_frac=0.5, redraw_p=0.1):
    """PRL records (SURVEY D-5): 8 u32 fields (Zipf(1.1) name codes folded into their
    domain, uniform otherwise), db_id = 1e9 + permutation(I); new records are 50 %
    noisy copies of random DB records (each field re-drawn with p = 0.1), 50 % fresh."""
    g_db, g_new, g_id = rng(seed_base + 1), rng(seed_base + 2), rng(seed_base + 3)

    def draw(g, n):
        cols = []
        for k, dom in enumerate(S.PRL_DOMAINS):
            if k < 3:
                cols.append(_zipf_codes(g, n, dom))
            else:
                cols.append(g.integers(0, dom, size=n, dtype=np.int64).astype(np.uint32))
        return cols

    db = draw(g_db, I)
    fresh = draw(g_new, N)
    src = g_new.integers(0, I, size=N)
    is_dup = g_new.random(N) < dup_frac
    new = []
    for k in range(S.PRL_FIELDS):
        col = np.where(is_dup, db[k][src], fresh[k]).astype(np.uint32)
        redraw = is_dup & (g_new.random(N) < redraw_p)
        repl = draw(g_new, N)[k]
        col = np.where(redraw, repl, col).astype(np.uint32)
        new.append(np.ascontiguousarray(col))
    db_id = (10 ** 9 + g_id.permutation(I)).astype(np.int64)
    return new + [np.ascontiguousarray(c) for c in db] + [db_id]


def prl_tiny():
    """The hand-made 3 new × 4 DB instance of SURVEY §8(c).5 (weights wa=[1..8], wd=-0.5)."""
    dbr = [list(range(1, 9)), [1, 2, 3, 4, 5, 6, 7, 9], [9] * 8, list(range(1, 9))]
    ids = [100, 101, 102, 103]
    newr = [list(range(1, 9)), [9, 9, 9, 9, 9, 9, 9, 0], [0] * 8]
    new = [np.array([r[k] for r in newr], np.uint32) for k in range(8)]
    db = [np.array([r[k] for r in dbr], np.uint32) for k in range(8)]
    wa = [float(k) for k in range(1, 9)]
    wd = [-0.5] * 8
    return new + db + [np.array(ids, np.int64)], (wa, wd)
