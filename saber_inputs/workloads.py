"""Query specifications (plain dicts) for the BASELINE.json configs.

A spec is the *text* of a windowed query -- nothing here evaluates it.

spec = {
  "schema":  {"tuple_bytes": B, "ts": "ts", "cols": [(name, type, offset), ...]},
  "window":  {"kind": "count"|"time", "size": s, "slide": l, "origin": T0},
  "where":   [(col, op, const), ...]          # conjunction; op in < <= > >= == !=
  "project": [col, ...]                       # σ/π (IStream) queries only
  "aggs":    [(fn, col), ...]                 # fn in sum count avg min max (RStream)
  "group_by":[(col, div, domain), ...]        # key = col / div; domain>0 declares [0,domain)
  "having":  [(agg_index, op, const), ...]
}

gen = {"kind": "syn"|"cm"|"sg"|"lrb", "n": tuples, "seed": s, "rate": R, "groups": G}

Config ids follow SURVEY.md §8 (C1..C5b) and BASELINE.json ``configs``.
"""
from __future__ import annotations

import copy

from .gen import SCHEMAS


def _spec(stream, window, where=(), project=(), aggs=(), group_by=(), having=()):
    return {
        "schema": copy.deepcopy(SCHEMAS[stream]),
        "window": dict(window),
        "where": [tuple(p) for p in where],
        "project": list(project),
        "aggs": [tuple(a) for a in aggs],
        "group_by": [tuple(k) for k in group_by],
        "having": [tuple(h) for h in having],
    }


def count_window(size, slide):
    return {"kind": "count", "size": int(size), "slide": int(slide), "origin": 0}


def time_window(size, slide, origin=0):
    return {"kind": "time", "size": int(size), "slide": int(slide), "origin": int(origin)}


# --- C1: SELECT SUM(a1) FROM Syn [ROWS 1024 SLIDE 1024] (configs[0]) -------------
def c1(fn="sum", n=1 << 20):
    return (_spec("syn", count_window(1024, 1024), aggs=[(fn, "a1")]),
            {"kind": "syn", "n": n, "seed": 1, "rate": 1, "groups": 64})


# --- C2: SELECT ts,a1,a2 FROM Syn [ROWS 1024 SLIDE 64] WHERE a3 < θ (configs[1]) --
def c2(sel=0.5, npred=1, n=1 << 25):
    theta = int(round(sel * 2 ** 31))
    where = [("a3", "<", theta)]
    extra = ["a4", "a5", "a6", "a2"]
    for k in range(npred - 1):          # always-true terms: same selectivity, more ALU (SELECT_n, Fig. 10a)
        where.append((extra[k % len(extra)], ">=", -k))
    return (_spec("syn", count_window(1024, 64), where=where, project=["ts", "a1", "a2"]),
            {"kind": "syn", "n": n, "seed": 2, "rate": 1, "groups": 64})


# --- C3: SELECT AVG(a1) FROM Syn [ROWS 32768 SLIDE 1024] GROUP BY a2 (configs[2]) --
def c3(groups=64, n=1 << 28, declare_domain=True):
    return (_spec("syn", count_window(32768, 1024), aggs=[("avg", "a1")],
                  group_by=[("a2", 1, groups if declare_domain else 0)]),
            {"kind": "syn", "n": n, "seed": 3, "rate": 1, "groups": groups})


# --- C4: CM1 SELECT SUM(cpu) FROM TaskEvents [RANGE 60 SLIDE 1] GROUP BY category --
def c4(rate=64, gcat=4, n=1 << 27, declare_domain=True):
    return (_spec("cm", time_window(60, 1), aggs=[("sum", "cpu")],
                  group_by=[("category", 1, gcat if declare_domain else 0)]),
            {"kind": "cm", "n": n, "seed": 4, "rate": rate, "groups": gcat})


# --- C5a: SG2 AVG(value) [RANGE 3600 SLIDE 1] GROUP BY plug, household, house ----
def c5a(n=1 << 28, rate=4096, declare_domain=True):
    d = declare_domain
    return (_spec("sg", time_window(3600, 1), aggs=[("avg", "value")],
                  group_by=[("plug", 1, 8 if d else 0), ("household", 1, 8 if d else 0),
                            ("house", 1, 32 if d else 0)]),
            {"kind": "sg", "n": n, "seed": 5, "rate": rate, "groups": 2048})


def sg1(n=1 << 28, rate=4096):
    return (_spec("sg", time_window(3600, 1), aggs=[("avg", "value")]),
            {"kind": "sg", "n": n, "seed": 5, "rate": rate, "groups": 2048})


# --- C5b: LRB3 AVG(speed) [RANGE 300 SLIDE 1] GROUP BY highway, direction,
#          position/5280 HAVING AVG(speed) < 40.0 ----------------------------------
def c5b(n=1 << 28, rate=8192, declare_domain=True):
    d = declare_domain
    return (_spec("lrb", time_window(300, 1), aggs=[("avg", "speed")],
                  group_by=[("highway", 1, 8 if d else 0), ("direction", 1, 2 if d else 0),
                            ("position", 5280, 100 if d else 0)],
                  having=[(0, "<", 40.0)]),
            {"kind": "lrb", "n": n, "seed": 6, "rate": rate, "groups": 0})


# --- f1 (next): CM2 avg(cpu) where eventType == 1 group by jobId (int64 key) -------
def cm2(rate=64, n=1 << 27):
    return (_spec("cm", time_window(60, 1), where=[("eventType", "==", 1)],
                  aggs=[("avg", "cpu")], group_by=[("jobId", 1, 0)]),
            {"kind": "cm", "n": n, "seed": 4, "rate": rate, "groups": 4})


CONFIGS = {"C1": c1, "C2": c2, "C3": c3, "C4": c4, "C5a": c5a, "C5b": c5b, "SG1": sg1, "CM2": cm2}


# Task size φ (MiB) bench.py uses per config (device-resident leg): the B200
# plateau of DESIGN.md §8, bounded where one task's result rows must fit a slot.
BENCH_TASK_MB = {"C1": 32, "C2": 1024, "C3": 4096, "C3_G256": 4096, "C3_G1024": 4096, "C3_G4096": 2048,
                 "C3_G16384": 512, "C3_G65536": 256, "C4": 4096, "C5a": 4096, "C5b": 4096, "SG1": 4096,
                 "CM2": 1024}


def bench_task_mb(config, groups=64):
    """φ in MiB for ``config`` (C3 depends on the group count)."""
    if config == "C3" and groups != 64:
        return BENCH_TASK_MB.get(f"C3_G{groups}", 1024 if groups <= 4096 else 256)
    return BENCH_TASK_MB[config]


# --- f3: JOIN_r, windowed θ-join of two Syn streams (Table 1, §6.2) ---
def join_r(r=1, size=1024, slide=1024, n=1 << 20):
    """SELECT S1.ts, S1.a1, S2.a1, S2.a2 FROM Syn1 [ROWS size SLIDE slide] AS S1,
    Syn2 [ROWS size SLIDE slide] AS S2 WHERE S1.a3 < S2.a3 AND S1.a4 < S2.a4 ...
    (r terms over a3..a6, cycling): the r-predicate θ-join JOIN_r; the attributes
    are uniform and independent, so 2^-min(r, 4) of the pairs match."""
    cols = ["a3", "a4", "a5", "a6"]
    theta = [(cols[k % 4], "<", cols[k % 4]) for k in range(r)]
    spec = {"schema1": copy.deepcopy(SCHEMAS["syn"]), "schema2": copy.deepcopy(SCHEMAS["syn"]),
            "window": count_window(size, slide), "theta": theta,
            "project1": ["ts", "a1"], "project2": ["a1", "a2"]}
    return spec, {"kind": "syn", "n": n, "seed1": 7, "seed2": 8, "rate": 1, "groups": 64}
