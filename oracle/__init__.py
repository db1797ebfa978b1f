"""TEST INFRASTRUCTURE ONLY -- the CPU oracle for a windowed streaming query.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_sigmod_koliousiswfwcp16_b200`` never imports it,
and this package never imports the product.  Both consume the same neutral
inputs from ``saber_inputs`` (generators + query spec dicts).

``liboracle.so`` (oracle.cpp) is the plain definition of PAPER.md §2.4
(L343-405): every closed window is enumerated and recomputed from scratch.
``brute.py`` is an independent pure-Python formulation used only to check
the C++ oracle on tiny inputs.  Readings of the paper are listed in
DESIGN.md §3; functions without an independent pin would be marked
"parity unpinned" here and in DESIGN.md (time-window extent A1, the output
timestamp A7 and empty-window headers A6 are fixed by reading, not by the
paper: see tests/test_oracle_pins.py for what pins what).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")

TYPES = {"i32": 0, "i64": 1, "f32": 2, "f64": 3}
OPS = {"<": 0, "<=": 1, ">": 2, ">=": 3, "==": 4, "!=": 5}
FNS = {"sum": 0, "count": 1, "avg": 2, "min": 3, "max": 4}


class _Col(C.Structure):
    _fields_ = [("off", C.c_int32), ("type", C.c_int32)]


class _Pred(C.Structure):
    _fields_ = [("off", C.c_int32), ("type", C.c_int32), ("op", C.c_int32), ("pad", C.c_int32),
                ("ival", C.c_int64), ("fval", C.c_double)]


class _Agg(C.Structure):
    _fields_ = [("fn", C.c_int32), ("off", C.c_int32), ("type", C.c_int32), ("pad", C.c_int32)]


class _Key(C.Structure):
    _fields_ = [("off", C.c_int32), ("type", C.c_int32), ("div", C.c_int64)]


class _Have(C.Structure):
    _fields_ = [("agg", C.c_int32), ("op", C.c_int32), ("ival", C.c_int64), ("fval", C.c_double)]


class _Query(C.Structure):
    _fields_ = [("tuple_bytes", C.c_int32), ("ts_off", C.c_int32),
                ("win_kind", C.c_int32), ("pad", C.c_int32),
                ("size", C.c_int64), ("slide", C.c_int64), ("origin", C.c_int64),
                ("npred", C.c_int32), ("pred", _Pred * 64),
                ("nproj", C.c_int32), ("proj", _Col * 16),
                ("nagg", C.c_int32), ("agg", _Agg * 8),
                ("nkeys", C.c_int32), ("key", _Key * 4),
                ("nhave", C.c_int32), ("have", _Have * 8)]


class _Result(C.Structure):
    _fields_ = [("error", C.c_int32), ("nwin", C.c_int64),
                ("win_id", C.POINTER(C.c_int64)), ("win_ts", C.POINTER(C.c_int64)),
                ("win_nrows", C.POINTER(C.c_int64)), ("win_rowoff", C.POINTER(C.c_int64)),
                ("nrows", C.c_int64), ("keys", C.POINTER(C.c_int64)),
                ("vals", C.POINTER(C.c_uint64)), ("val_is_float", C.c_int32 * 8),
                ("out_bytes", C.c_int64), ("out", C.POINTER(C.c_uint8)),
                ("row_bytes", C.c_int64)]


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain g++, no fast-math, no FP contraction)."""
    src = os.path.join(_HERE, "oracle.cpp")
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < max(
            os.path.getmtime(src), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-fPIC", "-shared", "-pthread",
                               "-ffp-contract=off", "-fno-fast-math", src, "-o", _SO + ".tmp"])
        os.replace(_SO + ".tmp", _SO)
    return _SO


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        _lib = C.CDLL(_SO)
        _lib.oq_run.restype = C.c_int32
        _lib.oq_run.argtypes = [C.POINTER(_Query), C.c_void_p, C.c_int64, C.c_int64, C.c_int32,
                                C.POINTER(C.c_int64), C.c_int64, C.c_int32, C.POINTER(_Result)]
        _lib.oq_num_windows.restype = C.c_int64
        _lib.oq_num_windows.argtypes = [C.POINTER(_Query), C.c_void_p, C.c_int64, C.c_int64, C.c_int32]
        _lib.oq_free.argtypes = [C.POINTER(_Result)]
        _lib.oq_join_run.restype = C.c_int32
        _lib.oq_join_run.argtypes = [C.POINTER(_Join), C.c_void_p, C.c_int64, C.c_void_p, C.c_int64, C.c_int32,
                                     C.POINTER(_Result)]
    return _lib


def _colinfo(spec, name):
    for cname, ctype, off in spec["schema"]["cols"]:
        if cname == name:
            return off, TYPES[ctype]
    raise KeyError(name)


def _marshal(spec) -> _Query:
    q = _Query()
    sch = spec["schema"]
    q.tuple_bytes = sch["tuple_bytes"]
    q.ts_off = _colinfo(spec, sch["ts"])[0]
    w = spec["window"]
    q.win_kind = 0 if w["kind"] == "count" else 1
    q.size, q.slide, q.origin = w["size"], w["slide"], w.get("origin", 0)
    q.npred = len(spec.get("where", []))
    for i, (col, op, const) in enumerate(spec.get("where", [])):
        off, t = _colinfo(spec, col)
        q.pred[i].off, q.pred[i].type, q.pred[i].op = off, t, OPS[op]
        if t in (2, 3):
            q.pred[i].fval = float(const)
        else:
            q.pred[i].ival = int(const)
    q.nproj = len(spec.get("project", []))
    for i, col in enumerate(spec.get("project", [])):
        q.proj[i].off, q.proj[i].type = _colinfo(spec, col)
    q.nagg = len(spec.get("aggs", []))
    for i, (fn, col) in enumerate(spec.get("aggs", [])):
        q.agg[i].fn = FNS[fn]
        if col not in (None, "*"):
            q.agg[i].off, q.agg[i].type = _colinfo(spec, col)
        else:
            q.agg[i].off, q.agg[i].type = 0, 0
    q.nkeys = len(spec.get("group_by", []))
    for i, (col, div, _dom) in enumerate(spec.get("group_by", [])):
        off, t = _colinfo(spec, col)
        q.key[i].off, q.key[i].type, q.key[i].div = off, t, int(div)
    q.nhave = len(spec.get("having", []))
    for i, (agg, op, const) in enumerate(spec.get("having", [])):
        q.have[i].agg, q.have[i].op = agg, OPS[op]
        q.have[i].fval = float(const)
        q.have[i].ival = int(const) if float(const) == int(const) else 0
    return q


class _JPred(C.Structure):
    _fields_ = [("off1", C.c_int32), ("type1", C.c_int32), ("op", C.c_int32), ("off2", C.c_int32),
                ("type2", C.c_int32), ("pad", C.c_int32)]


class _Join(C.Structure):
    _fields_ = [("tuple_bytes1", C.c_int32), ("tuple_bytes2", C.c_int32), ("ts_off1", C.c_int32),
                ("pad", C.c_int32), ("size", C.c_int64), ("slide", C.c_int64),
                ("npred", C.c_int32), ("pred", _JPred * 64),
                ("nproj1", C.c_int32), ("proj1", _Col * 16),
                ("nproj2", C.c_int32), ("proj2", _Col * 16)]


class OracleError(RuntimeError):
    def __init__(self, code):
        super().__init__(f"oracle error {code}")
        self.code = code


def run(spec, data, watermark=None, windows=None, nthreads=1):
    """Evaluate ``spec`` over ``data`` (bytes / uint8 array of row-major tuples).

    Returns a dict: win_id, win_ts, win_nrows, win_rowoff (int64 arrays),
    keys (int64 [nrows, nkeys]), vals (list per aggregate: float64 or int64
    array), tuples (IStream bytes), row_bytes.
    """
    L = lib()
    q = _marshal(spec)
    buf = np.ascontiguousarray(np.frombuffer(data, dtype=np.uint8) if isinstance(data, (bytes, bytearray))
                               else np.asarray(data, dtype=np.uint8).reshape(-1))
    n = buf.size // q.tuple_bytes
    ids = None
    nids = 0
    if windows is not None:
        ids_arr = np.ascontiguousarray(np.asarray(windows, dtype=np.int64))
        ids = ids_arr.ctypes.data_as(C.POINTER(C.c_int64))
        nids = ids_arr.size
    res = _Result()
    err = L.oq_run(C.byref(q), buf.ctypes.data if buf.size else None, n,
                   0 if watermark is None else int(watermark), 0 if watermark is None else 1,
                   ids, nids, int(nthreads), C.byref(res))
    try:
        if err != 0:
            raise OracleError(err)
        nw, nr = res.nwin, res.nrows

        def arr(p, cnt, dt=np.int64):
            return np.ctypeslib.as_array(p, shape=(cnt,)).astype(dt).copy() if cnt else np.zeros(0, dt)
        out = {
            "win_id": arr(res.win_id, nw), "win_ts": arr(res.win_ts, nw),
            "win_nrows": arr(res.win_nrows, nw), "win_rowoff": arr(res.win_rowoff, nw),
        }
        nk, na = q.nkeys, q.nagg
        out["keys"] = arr(res.keys, nr * nk).reshape(nr, nk) if nk else np.zeros((nr, 0), np.int64)
        raw = (np.ctypeslib.as_array(res.vals, shape=(nr * na,)).copy() if nr * na
               else np.zeros(0, np.uint64)).reshape(nr, na) if na else np.zeros((nr, 0), np.uint64)
        out["vals"] = [raw[:, a].view(np.float64 if res.val_is_float[a] else np.int64).copy()
                       for a in range(na)]
        out["tuples"] = bytes(np.ctypeslib.as_array(res.out, shape=(res.out_bytes,))) if res.out_bytes else b""
        out["row_bytes"] = res.row_bytes
        return out
    finally:
        L.oq_free(C.byref(res))


def num_windows(spec, data, watermark=None):
    L = lib()
    q = _marshal(spec)
    buf = np.ascontiguousarray(np.frombuffer(data, dtype=np.uint8) if isinstance(data, (bytes, bytearray))
                               else np.asarray(data, dtype=np.uint8).reshape(-1))
    n = buf.size // q.tuple_bytes
    return L.oq_num_windows(C.byref(q), buf.ctypes.data if buf.size else None, n,
                            0 if watermark is None else int(watermark), 0 if watermark is None else 1)


def join_run(jspec, data1, data2, nthreads=1):
    """Windowed θ-join of two streams (oracle.h oq_join_run).  ``jspec``:
    schema1, schema2, window (count), theta [(col1, op, col2)], project1, project2.
    Returns win_id, win_ts, win_nrows, win_rowoff and ``tuples`` (pair rows)."""
    L = lib()
    q = _Join()
    s1, s2 = jspec["schema1"], jspec["schema2"]
    q.tuple_bytes1, q.tuple_bytes2 = s1["tuple_bytes"], s2["tuple_bytes"]
    q.ts_off1 = _colinfo({"schema": s1}, s1["ts"])[0]
    w = jspec["window"]
    q.size, q.slide = w["size"], w["slide"]
    q.npred = len(jspec.get("theta", []))
    for i, (c1, op, c2) in enumerate(jspec.get("theta", [])):
        q.pred[i].off1, q.pred[i].type1 = _colinfo({"schema": s1}, c1)
        q.pred[i].off2, q.pred[i].type2 = _colinfo({"schema": s2}, c2)
        q.pred[i].op = OPS[op]
    q.nproj1 = len(jspec["project1"])
    for i, c in enumerate(jspec["project1"]):
        q.proj1[i].off, q.proj1[i].type = _colinfo({"schema": s1}, c)
    q.nproj2 = len(jspec["project2"])
    for i, c in enumerate(jspec["project2"]):
        q.proj2[i].off, q.proj2[i].type = _colinfo({"schema": s2}, c)
    b1 = np.ascontiguousarray(np.frombuffer(data1, np.uint8) if isinstance(data1, (bytes, bytearray)) else data1)
    b2 = np.ascontiguousarray(np.frombuffer(data2, np.uint8) if isinstance(data2, (bytes, bytearray)) else data2)
    res = _Result()
    err = L.oq_join_run(C.byref(q), b1.ctypes.data if b1.size else None, b1.size // q.tuple_bytes1,
                        b2.ctypes.data if b2.size else None, b2.size // q.tuple_bytes2, int(nthreads), C.byref(res))
    try:
        if err != 0:
            raise OracleError(err)
        nw = res.nwin

        def arr(p, cnt):
            return np.ctypeslib.as_array(p, shape=(cnt,)).astype(np.int64).copy() if cnt else np.zeros(0, np.int64)
        return {"win_id": arr(res.win_id, nw), "win_ts": arr(res.win_ts, nw), "win_nrows": arr(res.win_nrows, nw),
                "win_rowoff": arr(res.win_rowoff, nw), "row_bytes": res.row_bytes,
                "tuples": bytes(np.ctypeslib.as_array(res.out, shape=(res.out_bytes,))) if res.out_bytes else b""}
    finally:
        L.oq_free(C.byref(res))
