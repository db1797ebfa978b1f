"""Tiny hand-built streams for the golden / brute-force tests.

Schema "tiny" (32-B tuples): ts i64 @0, v i32 @8, x f32 @12, m i64 @16
(m = 2^position: an integer SUM of m is the window's membership bitmask),
k i32 @24 (group key), o i32 @28 (1 if v is odd).
"""
import json
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")

TINY = {"tuple_bytes": 32, "ts": "ts", "cols": [
    ("ts", "i64", 0), ("v", "i32", 8), ("x", "f32", 12), ("m", "i64", 16),
    ("k", "i32", 24), ("o", "i32", 28)]}


def golden(name):
    for f in os.listdir(GOLDEN):
        if f.startswith(name + "_"):
            with open(os.path.join(GOLDEN, f)) as fh:
                return json.load(fh)
    raise KeyError(name)


def stream(v=None, tau=None, x=None, k=None, n=None):
    if n is None:
        n = len(next(a for a in (v, tau, x, k) if a is not None))
    a = np.zeros(n, dtype=[("ts", "<i8"), ("v", "<i4"), ("x", "<f4"), ("m", "<i8"),
                           ("k", "<i4"), ("o", "<i4")])
    a["ts"] = np.arange(n) if tau is None else tau
    if v is not None:
        a["v"] = v
        a["o"] = np.asarray(v) % 2
    if x is not None:
        a["x"] = x
    a["m"] = (np.int64(1) << np.arange(n, dtype=np.int64)) if n < 63 else 0
    if k is not None:
        a["k"] = k
    return a.tobytes()


def spec(window, where=(), project=(), aggs=(), group_by=(), having=()):
    return {"schema": TINY, "window": dict(window), "where": list(where), "project": list(project),
            "aggs": list(aggs), "group_by": list(group_by), "having": list(having)}
