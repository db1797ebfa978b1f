"""Cross-check the C++ oracle against the independent pure-Python brute force
(oracle/brute.py) on thousands of tiny random streams:
1 <= l <= s <= 8, N <= 40, G <= 4, time streams with gaps and runs of equal
timestamps, random selection thresholds, every aggregate, IStream.  Results
must be identical (floats included: both sum in increasing position order)."""
import numpy as np
import pytest

from oracle.brute import brute
from tiny import spec, stream


def _from_oracle(res, sp):
    out = []
    nk = len(sp["group_by"])
    for w in range(len(res["win_id"])):
        o, n = res["win_rowoff"][w], res["win_nrows"][w]
        if sp["aggs"]:
            rows = []
            for r in range(o, o + n):
                key = tuple(int(res["keys"][r][k]) for k in range(nk))
                vals = [v[r].item() for v in res["vals"]]
                rows.append((key, vals))
        else:
            rb = res["row_bytes"]
            rows = [res["tuples"][r * rb:(r + 1) * rb] for r in range(o, o + n)]
        out.append((int(res["win_id"][w]), int(res["win_ts"][w]), rows))
    return out


def _case(rng):
    n = int(rng.integers(0, 41))
    s = int(rng.integers(1, 9))
    l = int(rng.integers(1, s + 1))
    kind = "count" if rng.random() < 0.5 else "time"
    if kind == "time":
        steps = rng.choice([0, 0, 1, 1, 2, 3], size=n)
        tau = np.cumsum(steps) + int(rng.integers(0, 3))
    else:
        tau = np.arange(n)
    v = rng.integers(-20, 20, size=n)
    x = rng.integers(0, 64, size=n) / 8.0                    # dyadic: exact in f32 and f64
    k = rng.integers(0, int(rng.integers(1, 5)), size=n)
    where = []
    if rng.random() < 0.5:
        where.append(("v", rng.choice(["<", "<=", ">", ">=", "==", "!="]), int(rng.integers(-20, 20))))
    if rng.random() < 0.3:
        where.append(("x", rng.choice(["<", ">="]), float(rng.integers(0, 8))))
    w = {"kind": kind, "size": s, "slide": l, "origin": int(rng.integers(0, 2)) if kind == "time" else 0}
    if rng.random() < 0.25:
        sp = spec(w, where=where, project=list(rng.choice(["ts", "v", "x", "k"], size=int(rng.integers(1, 4)))))
    else:
        fns = ["sum", "count", "avg", "min", "max"]
        aggs = [(str(rng.choice(fns)), str(rng.choice(["v", "x"]))) for _ in range(int(rng.integers(1, 4)))]
        aggs = [(f, None) if f == "count" else (f, c) for f, c in aggs]
        gb = [("k", 1, 0)] if rng.random() < 0.6 else []
        if gb and rng.random() < 0.3:
            gb.append(("v", int(rng.choice([1, 3, -4])), 0))
        having = []
        if rng.random() < 0.3:
            a = int(rng.integers(0, len(aggs)))
            having.append((a, str(rng.choice(["<", ">="])), float(rng.integers(-5, 10))))
        sp = spec(w, where=where, aggs=aggs, group_by=gb, having=having)
    wm = None
    if kind == "time" and rng.random() < 0.3:
        wm = int((tau[-1] if n else 0) + rng.integers(0, 6))
    return sp, stream(v=v, tau=tau, x=x, k=k, n=n), wm


@pytest.mark.parametrize("seed", range(8))
def test_oracle_vs_brute(oracle_lib, seed):
    rng = np.random.default_rng(1000 + seed)
    for _ in range(300):
        sp, d, wm = _case(rng)
        res = oracle_lib.run(sp, d, watermark=wm)
        assert _from_oracle(res, sp) == brute(sp, d, watermark=wm), (sp, wm)
