"""TEST INFRASTRUCTURE ONLY -- an independent pure-Python brute force.

Used solely to check the C++ oracle (liboracle.so) on tiny streams.  It is
written differently on purpose: 1-based tuple indices as in the paper
(w_i = <t_k..t_m>, m = k+s-1, next window starts at t_{k+l}: PAPER.md
L370-372), time windows as a set-builder over *all* positions (no binary
search), per-window dict of groups, struct.unpack decoding.
"""
from __future__ import annotations

import struct

_FMT = {"i32": "<i", "i64": "<q", "f32": "<f", "f64": "<d"}
_W = {"i32": 4, "i64": 8, "f32": 4, "f64": 8}
_OPS = {"<": lambda a, b: a < b, "<=": lambda a, b: a <= b, ">": lambda a, b: a > b,
        ">=": lambda a, b: a >= b, "==": lambda a, b: a == b, "!=": lambda a, b: a != b}


def _col(spec, name):
    for c, t, off in spec["schema"]["cols"]:
        if c == name:
            return t, off
    raise KeyError(name)


def _get(spec, raw, name):
    t, off = _col(spec, name)
    return struct.unpack_from(_FMT[t], raw, off)[0]


def _trunc_div(a, b):
    q = abs(a) // abs(b)
    return q if (a >= 0) == (b > 0) else -q


def brute(spec, data, watermark=None):
    tb = spec["schema"]["tuple_bytes"]
    n = len(data) // tb
    t = [bytes(data[i * tb:(i + 1) * tb]) for i in range(n)]           # t[1..n] in the paper
    tau = [_get(spec, x, spec["schema"]["ts"]) for x in t]
    w = spec["window"]
    s, l = w["size"], w["slide"]
    wins = []                                                        # list of (j, [positions], ts)
    if w["kind"] == "count":
        k, j = 1, 0
        while True:
            m = k + s - 1
            if m > n:
                break
            wins.append((j, list(range(k - 1, m)), tau[k - 1]))
            k, j = k + l, j + 1
    else:
        T0 = w.get("origin", 0)
        wm = watermark if watermark is not None else (tau[-1] + 1 if n else None)
        j = 0
        while wm is not None and T0 + j * l + s <= wm:
            lo, hi = T0 + j * l, T0 + j * l + s
            wins.append((j, [i for i in range(n) if lo <= tau[i] < hi], lo))
            j += 1

    def sel(x):
        for col, op, c in spec.get("where", []):
            if not _OPS[op](_get(spec, x, col), c):
                return False
        return True

    result = []
    prev = set()
    for j, pos, ts in wins:
        if not spec.get("aggs"):
            rows = []
            for i in pos:
                if i not in prev and sel(t[i]):
                    rows.append(b"".join(t[i][_col(spec, c)[1]:_col(spec, c)[1] + _W[_col(spec, c)[0]]]
                                         for c in spec["project"]))
            result.append((j, ts, rows))
            prev = set(pos)
            continue
        groups = {}
        for i in pos:
            if not sel(t[i]):
                continue
            key = tuple(_trunc_div(_get(spec, t[i], c), d) for c, d, _ in spec.get("group_by", []))
            groups.setdefault(key, []).append(i)
        rows = []
        for key in sorted(groups):
            vals = []
            for fn, col in spec["aggs"]:
                xs = [_get(spec, t[i], col) for i in groups[key]] if col not in (None, "*") else []
                if fn == "count":
                    vals.append(len(groups[key]))
                elif fn == "sum":
                    acc = 0.0 if _col(spec, col)[0] in ("f32", "f64") else 0
                    for x in xs:
                        acc += x
                    vals.append(acc)
                elif fn == "avg":
                    acc = 0.0 if _col(spec, col)[0] in ("f32", "f64") else 0
                    for x in xs:
                        acc += x
                    vals.append(float(acc) / len(xs))
                elif fn == "min":
                    vals.append(min(xs))
                elif fn == "max":
                    vals.append(max(xs))
            if all(_OPS[op](vals[a], c) for a, op, c in spec.get("having", [])):
                rows.append((key, vals))
        result.append((j, ts, rows))
    return result


def brute_join(jspec, d1, d2):
    """Windowed θ-join, written independently of oracle.cpp: 1-based windows
    <t_k..t_m> on both streams (L370-372), a Python set of matching position
    pairs per window, rows sorted by (a, b) only at the end."""
    s1, s2 = jspec["schema1"], jspec["schema2"]
    n1, n2 = len(d1) // s1["tuple_bytes"], len(d2) // s2["tuple_bytes"]
    t1 = [bytes(d1[i * s1["tuple_bytes"]:(i + 1) * s1["tuple_bytes"]]) for i in range(n1)]
    t2 = [bytes(d2[i * s2["tuple_bytes"]:(i + 1) * s2["tuple_bytes"]]) for i in range(n2)]
    sp1, sp2 = {"schema": s1}, {"schema": s2}
    w = jspec["window"]
    s, l = w["size"], w["slide"]
    out = []
    k, j = 1, 0
    while k + s - 1 <= min(n1, n2):
        pos = range(k - 1, k + s - 1)
        pairs = set()
        for a in pos:
            for b in pos:
                ok = True
                for c1, op, c2 in jspec.get("theta", []):
                    x, y = _get(sp1, t1[a], c1), _get(sp2, t2[b], c2)
                    if not _OPS[op](x, y):
                        ok = False
                        break
                if ok:
                    pairs.add((a, b))
        rows = []
        for a, b in sorted(pairs):
            r = b"".join(t1[a][_col(sp1, c)[1]:_col(sp1, c)[1] + _W[_col(sp1, c)[0]]] for c in jspec["project1"])
            r += b"".join(t2[b][_col(sp2, c)[1]:_col(sp2, c)[1] + _W[_col(sp2, c)[0]]] for c in jspec["project2"])
            rows.append(r)
        out.append((j, _get(sp1, t1[k - 1], s1["ts"]), rows))
        k, j = k + l, j + 1
    return out
