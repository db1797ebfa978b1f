"""Counter-based synthetic stream generator (host side, numpy).

The formulas are SURVEY.md §8(d) D1; the layouts follow the paper:

* Syn: 32-B tuples, int64 timestamp + six 32-bit
  attributes, uniform, "the first value being a float".
* CM   (App. A.1): 64-B TaskEvents.
* SG   (App. A.2): 32-B SmartGridStr.
* LRB  (App. A.3): 32-B PosSpeedStr.

Every byte of tuple ``i`` depends only on ``(seed, i, params)``, so any slice
``[i0, i0+n)`` can be generated independently -- by this module or by the
device generator in ``csrc/gen.cu`` (which must produce identical bytes; a GPU
test checks that).  Timestamps are ``ts = i // rate`` (rate=1 gives ts = i,
the count-based configs' choice that makes time windows over them equal to
count windows).
"""
from __future__ import annotations

import numpy as np

U64 = np.uint64
_GOLD = U64(0x9E3779B97F4A7C15)
_M1 = U64(0xBF58476D1CE4E5B9)
_M2 = U64(0x94D049BB133111EB)

# (name, type, byte offset) -- type in {"i32","i64","f32","f64"}
SCHEMAS = {
    "syn": dict(tuple_bytes=32, ts="ts", cols=[
        ("ts", "i64", 0), ("a1", "f32", 8), ("a2", "i32", 12), ("a3", "i32", 16),
        ("a4", "i32", 20), ("a5", "i32", 24), ("a6", "i32", 28)]),
    "cm": dict(tuple_bytes=64, ts="ts", cols=[
        ("ts", "i64", 0), ("jobId", "i64", 8), ("taskId", "i64", 16),
        ("machineId", "i64", 24), ("eventType", "i32", 32), ("userId", "i32", 36),
        ("category", "i32", 40), ("priority", "i32", 44), ("cpu", "f32", 48),
        ("ram", "f32", 52), ("disk", "f32", 56), ("constraints", "i32", 60)]),
    "sg": dict(tuple_bytes=32, ts="ts", cols=[
        ("ts", "i64", 0), ("value", "f32", 8), ("property", "i32", 12),
        ("plug", "i32", 16), ("household", "i32", 20), ("house", "i32", 24),
        ("padding", "i32", 28)]),
    "lrb": dict(tuple_bytes=32, ts="ts", cols=[
        ("ts", "i64", 0), ("vehicle", "i32", 8), ("speed", "f32", 12),
        ("highway", "i32", 16), ("lane", "i32", 20), ("direction", "i32", 24),
        ("position", "i32", 28)]),
}

KIND_ID = {"syn": 0, "cm": 1, "sg": 2, "lrb": 3}


def splitmix64(z: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = z + _GOLD
        z = (z ^ (z >> U64(30))) * _M1
        z = (z ^ (z >> U64(27))) * _M2
        return z ^ (z >> U64(31))


def r(seed: int, i: np.ndarray, c: int) -> np.ndarray:
    return splitmix64((U64(seed) << U64(48)) ^ (i << U64(4)) ^ U64(c))


def u24(x):  # [0,1), exact in f32, never -0.0 / NaN
    return (x >> U64(40)).astype(np.float32) * np.float32(2.0 ** -24)


def u24_f64(x):
    return (x >> U64(40)).astype(np.float64) * (2.0 ** -24)


def u31(x):
    return (x >> U64(33)).astype(np.int32)


def uG(x, G: int):
    return ((x >> U64(32)) % U64(G)).astype(np.int32)


def generate(kind: str, n: int, seed: int, i0: int = 0, rate: int = 1,
             groups: int = 64) -> bytes:
    """Return ``n`` tuples (row-major bytes) of stream ``kind`` starting at
    global tuple index ``i0``.  ``groups`` is G for Syn's a2 / CM's category."""
    return generate_array(kind, n, seed, i0, rate, groups).tobytes()


def generate_array(kind: str, n: int, seed: int, i0: int = 0, rate: int = 1,
                   groups: int = 64) -> np.ndarray:
    sch = SCHEMAS[kind]
    tb = sch["tuple_bytes"]
    out = np.zeros((n, tb), dtype=np.uint8)
    if n == 0:
        return out
    i = np.arange(i0, i0 + n, dtype=np.uint64)
    ts = (i // U64(rate)).astype(np.int64)

    def put(off, arr):
        a = np.ascontiguousarray(arr)
        w = a.dtype.itemsize
        out[:, off:off + w] = a.view(np.uint8).reshape(n, w)

    put(0, ts)
    if kind == "syn":
        put(8, u24(r(seed, i, 1)))
        put(12, uG(r(seed, i, 2), groups))
        for c, off in zip(range(3, 7), (16, 20, 24, 28)):
            put(off, u31(r(seed, i, c)))
    elif kind == "cm":
        put(8, ((r(seed, i, 1) >> U64(32)) % U64(1 << 16)).astype(np.int64))
        put(16, u31(r(seed, i, 2)).astype(np.int64))
        put(24, u31(r(seed, i, 3)).astype(np.int64))
        put(32, ((r(seed, i, 4) >> U64(32)) % U64(9)).astype(np.int32))
        put(36, u31(r(seed, i, 5)))
        put(40, uG(r(seed, i, 6), groups))
        put(44, u31(r(seed, i, 7)))
        put(48, u24(r(seed, i, 8)))
        put(52, u24(r(seed, i, 9)))
        put(56, u24(r(seed, i, 10)))
        put(60, u31(r(seed, i, 11)))
    elif kind == "sg":
        put(8, u24(r(seed, i, 1)) * np.float32(1000.0))
        put(12, (r(seed, i, 2) & U64(1)).astype(np.int32))
        k = uG(r(seed, i, 3), 2048)
        put(16, k & 7)
        put(20, (k >> 3) & 7)
        put(24, k >> 6)
        put(28, np.zeros(n, dtype=np.int32))
    elif kind == "lrb":
        hwy = uG(r(seed, i, 3), 8)
        lane = uG(r(seed, i, 4), 4)
        dirn = uG(r(seed, i, 5), 2)
        pos = ((r(seed, i, 6) >> U64(32)) % U64(528000)).astype(np.int32)
        seg = pos // 5280
        base = np.where((hwy * 200 + dirn * 100 + seg) % 4 == 0, 30.0, 60.0)
        speed = (base - 10.0 + 20.0 * u24_f64(r(seed, i, 2))).astype(np.float32)
        put(8, (u31(r(seed, i, 1)) % (1 << 17)).astype(np.int32))
        put(12, speed)
        put(16, hwy)
        put(20, lane)
        put(24, dirn)
        put(28, pos)
    else:
        raise ValueError(kind)
    return out


def column(data: bytes | np.ndarray, kind_or_schema, name: str) -> np.ndarray:
    """Decode one column of a generated stream (test convenience)."""
    sch = SCHEMAS[kind_or_schema] if isinstance(kind_or_schema, str) else kind_or_schema
    tb = sch["tuple_bytes"]
    arr = np.frombuffer(data, dtype=np.uint8) if isinstance(data, (bytes, bytearray)) else data.reshape(-1)
    arr = arr.reshape(-1, tb)
    for cname, ctype, off in sch["cols"]:
        if cname == name:
            dt = {"i32": np.int32, "i64": np.int64, "f32": np.float32, "f64": np.float64}[ctype]
            w = np.dtype(dt).itemsize
            return np.ascontiguousarray(arr[:, off:off + w]).view(dt).reshape(-1)
    raise KeyError(name)


def wide_f32(seed: int, i0: int, n: int, lo_exp: float = -6.0, hi_exp: float = 12.0) -> np.ndarray:
    """Non-negative, non-dyadic f32 values spanning 10^lo_exp .. 10^hi_exp
    (log-uniform, counter-based): the float-robustness stream of DESIGN.md §4.
    fp64 sums of these are NOT exact, unlike u24 data."""
    i = np.arange(i0, i0 + n, dtype=np.uint64)
    u = u24_f64(r(seed, i, 13)) + u24_f64(r(seed, i, 14)) * 2.0 ** -24
    return (10.0 ** (lo_exp + (hi_exp - lo_exp) * u)).astype(np.float32)


def with_column(data: bytes, kind: str, name: str, values: np.ndarray) -> bytes:
    """Return ``data`` with column ``name`` replaced by ``values`` (test inputs)."""
    sch = SCHEMAS[kind]
    tb = sch["tuple_bytes"]
    arr = np.frombuffer(data, dtype=np.uint8).reshape(-1, tb).copy()
    for cname, ctype, off in sch["cols"]:
        if cname == name:
            v = np.ascontiguousarray(values.astype({"f32": np.float32, "i32": np.int32, "i64": np.int64,
                                                    "f64": np.float64}[ctype]))
            arr[:, off:off + v.itemsize] = v.view(np.uint8).reshape(-1, v.itemsize)
            return arr.tobytes()
    raise KeyError(name)
