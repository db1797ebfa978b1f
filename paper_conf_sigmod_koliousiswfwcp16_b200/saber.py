"""Thin ctypes binding of include/saber.h (argument marshalling only).

Every step of a query task runs in ``libsaber.so``'s sm_100a kernels; this
module only builds the C structs, calls the C ABI and copies finished result
slices into numpy arrays.  If the library is missing or there is no CUDA
device, calls fail loudly -- there is no CPU fallback.

Query specs are the plain dicts of ``saber_inputs.workloads`` (the text of a
query: schema, window, where, project, aggs, group_by, having).
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# SABER_LIB: an alternative build of the same sources (tuning experiments, scripts/build_variant.sh)
LIB_PATH = os.environ.get("SABER_LIB") or os.path.join(_HERE, "libsaber.so")

OK, EINVAL, ENOMEM, EAGAIN = 0, -22, -12, -11
EORDER, ECUDA, ENCCL, ECLOSED, ETS, EKEY, ECAPACITY = -1001, -1002, -1003, -1004, -1005, -1006, -1007
STATUS_NAMES = {0: "OK", -22: "EINVAL", -12: "ENOMEM", -11: "EAGAIN", -1001: "EORDER", -1002: "ECUDA",
                -1003: "ENCCL", -1004: "ECLOSED", -1005: "ETS", -1006: "EKEY", -1007: "ECAPACITY"}
TYPES = {"i32": 0, "i64": 1, "f32": 2, "f64": 3}
OPS = {"<": 0, "<=": 1, ">": 2, ">=": 3, "==": 4, "!=": 5}
FNS = {"sum": 0, "count": 1, "avg": 2, "min": 3, "max": 4}
RESULTS_HOST, RESULTS_DEVICE = 0, 1


class SaberError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


class Schema(C.Structure):
    _fields_ = [("ncols", C.c_int32), ("types", C.POINTER(C.c_int32)), ("offsets", C.POINTER(C.c_int32)),
                ("tuple_bytes", C.c_int32), ("ts_col", C.c_int32)]


class Window(C.Structure):
    _fields_ = [("kind", C.c_int32), ("size", C.c_int64), ("slide", C.c_int64), ("origin", C.c_int64)]


class Pred(C.Structure):
    _fields_ = [("col", C.c_int32), ("op", C.c_int32), ("ival", C.c_int64), ("fval", C.c_double)]


class Agg(C.Structure):
    _fields_ = [("fn", C.c_int32), ("col", C.c_int32)]


class KeyExpr(C.Structure):
    _fields_ = [("col", C.c_int32), ("div", C.c_int32), ("domain", C.c_int64)]


class Operator(C.Structure):
    _fields_ = [("npred", C.c_int32), ("where", C.POINTER(Pred)), ("nproj", C.c_int32),
                ("proj", C.POINTER(C.c_int32)), ("nagg", C.c_int32), ("aggs", C.POINTER(Agg)),
                ("nkeys", C.c_int32), ("group_by", C.POINTER(KeyExpr)), ("nhave", C.c_int32),
                ("having", C.POINTER(Pred))]


class Config(C.Structure):
    _fields_ = [("device", C.c_int32), ("task_bytes", C.c_int64), ("pipeline_depth", C.c_int32),
                ("result_mode", C.c_int32), ("result_bytes", C.c_int64), ("hash_capacity", C.c_int64),
                ("max_panes", C.c_int64), ("base_index", C.c_int64), ("first_window", C.c_int64),
                ("emit_on_finish", C.c_int32), ("result_slots", C.c_int32), ("profile", C.c_int32),
                ("reserved", C.c_int32 * 5)]


class WinHdr(C.Structure):
    _fields_ = [("window_id", C.c_int64), ("ts", C.c_int64), ("row_offset", C.c_int64),
                ("nrows", C.c_int32), ("flags", C.c_int32)]


class Results(C.Structure):
    _fields_ = [("task_id", C.c_int64), ("first_window", C.c_int64), ("nwindows", C.c_int64),
                ("hdr", C.POINTER(WinHdr)), ("nrows", C.c_int64), ("ncols", C.c_int32),
                ("on_device", C.c_int32), ("cols", C.c_void_p * 12), ("col_bytes", C.c_int32 * 12),
                ("tuples", C.c_void_p), ("tuple_bytes", C.c_int32), ("reserved", C.c_int32),
                ("ntuples", C.c_int64)]


class Stats(C.Structure):
    _fields_ = [("tasks", C.c_int64), ("tuples", C.c_int64), ("bytes_in", C.c_int64), ("windows", C.c_int64),
                ("rows", C.c_int64), ("out_tuples", C.c_int64), ("tasks_pending", C.c_int64),
                ("last_complete", C.c_int64), ("last_opening", C.c_int64), ("last_closing", C.c_int64),
                ("last_pending", C.c_int64), ("kernel_launches", C.c_int64), ("scan_launches", C.c_int64),
                ("scan_ms", C.c_double), ("assemble_ms", C.c_double), ("scan_kind", C.c_int32),
                ("window_kind", C.c_int32), ("scan_grid", C.c_int32), ("window_grid", C.c_int32),
                ("overlap", C.c_int32), ("reserved", C.c_int32), ("task_tuples", C.c_int64)]

SCAN_KERNELS = ["k_select", "k_pane_agg", "k_pane_cnt", "k_pane_bucket"]
WINDOW_KERNELS = ["none", "k_vh_build+k_win_packed/k_win_fused", "k_win_block (or k_wb_rows+k_win_block_reg)",
                  "k_bkt_rows/k_bkt_count+k_win_scan+k_bkt_emit",
                  "k_win_hash", "k_win_slab", "k_vh_build+k_win_wide"]


# every function declared in include/saber.h: name -> (restype, argtypes)
SIGNATURES = {
    "saber_query_create": (C.c_int, [C.POINTER(Schema), C.POINTER(Operator), C.POINTER(Window),
                                     C.POINTER(Config), C.POINTER(C.c_void_p)]),
    "saber_task_submit": (C.c_int, [C.c_void_p, C.c_void_p, C.c_size_t]),
    "saber_task_submit_device": (C.c_int, [C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p]),
    "saber_register_host": (C.c_int, [C.c_void_p, C.c_void_p, C.c_size_t]),
    "saber_query_finish": (C.c_int, [C.c_void_p, C.c_int64]),
    "saber_results_poll": (C.c_int, [C.c_void_p, C.POINTER(Results), C.c_int32]),
    "saber_results_release": (C.c_int, [C.c_void_p, C.POINTER(Results)]),
    "saber_query_stats": (C.c_int, [C.c_void_p, C.POINTER(Stats)]),
    "saber_query_sync": (C.c_int, [C.c_void_p]),
    "saber_query_record": (C.c_int, [C.c_void_p, C.c_void_p]),
    "saber_query_reset": (C.c_int, [C.c_void_p, C.c_int64, C.c_int64]),
    "saber_query_destroy": (None, [C.c_void_p]),
    "saber_last_error": (C.c_char_p, [C.c_void_p]),
    "saber_partition_plan": (C.c_int, [C.POINTER(Schema), C.POINTER(Window), C.c_void_p, C.c_int64, C.c_int64,
                                       C.POINTER(C.c_int64), C.POINTER(C.c_int64)]),
    "saber_version": (C.c_char_p, []),
    "saber_join_create": (C.c_int, [C.POINTER(Schema), C.POINTER(Schema), C.c_void_p, C.POINTER(Window),
                                    C.POINTER(Config), C.POINTER(C.c_void_p)]),
    "saber_join_submit_device": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p]),
    "saber_join_submit": (C.c_int, [C.c_void_p, C.c_void_p, C.c_void_p, C.c_size_t]),
    "saber_join_poll": (C.c_int, [C.c_void_p, C.POINTER(Results), C.c_int32]),
    "saber_join_release": (C.c_int, [C.c_void_p, C.POINTER(Results)]),
    "saber_join_destroy": (None, [C.c_void_p]),
    "saber_join_last_error": (C.c_char_p, [C.c_void_p]),
}


class JoinPred(C.Structure):
    _fields_ = [("col1", C.c_int32), ("op", C.c_int32), ("col2", C.c_int32)]


class JoinOp(C.Structure):
    _fields_ = [("npred", C.c_int32), ("theta", C.POINTER(JoinPred)), ("nproj1", C.c_int32),
                ("proj1", C.POINTER(C.c_int32)), ("nproj2", C.c_int32), ("proj2", C.POINTER(C.c_int32))]

_lib = None


def lib():
    """Load libsaber.so (built in-tree by __graft_entry__.build()).  Fails loudly."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                              "(there is no CPU fallback for the SABER hot path)")
        L = C.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def _check(status, q=None):
    if status != OK:
        msg = lib().saber_last_error(q)
        raise SaberError(status, msg.decode() if msg else "")


class _Marshalled:
    """Keeps the ctypes arrays referenced by the C structs alive."""

    def __init__(self, spec):
        sch = spec["schema"]
        cols = sch["cols"]
        self.names = [c[0] for c in cols]
        self.types = (C.c_int32 * len(cols))(*[TYPES[c[1]] for c in cols])
        self.offsets = (C.c_int32 * len(cols))(*[c[2] for c in cols])
        self.schema = Schema(len(cols), self.types, self.offsets, sch["tuple_bytes"], self.names.index(sch["ts"]))
        w = spec["window"]
        self.window = Window(0 if w["kind"] == "count" else 1, w["size"], w["slide"], w.get("origin", 0))
        ctype = {c[0]: c[1] for c in cols}

        def pred(col, op, const, is_float):
            return Pred(col, OPS[op], int(const) if not is_float else 0, float(const))
        where = spec.get("where", [])
        self.where = (Pred * max(1, len(where)))(*[
            pred(self.names.index(c), op, v, ctype[c] in ("f32", "f64")) for c, op, v in where])
        proj = spec.get("project", [])
        self.proj = (C.c_int32 * max(1, len(proj)))(*[self.names.index(c) for c in proj])
        aggs = spec.get("aggs", [])
        self.aggs = (Agg * max(1, len(aggs)))(*[
            Agg(FNS[fn], self.names.index(col) if col not in (None, "*") else 0) for fn, col in aggs])
        gb = spec.get("group_by", [])
        self.keys = (KeyExpr * max(1, len(gb)))(*[KeyExpr(self.names.index(c), int(d), int(dom)) for c, d, dom in gb])
        hv = spec.get("having", [])

        def hpred(a, op, const):
            fn, col = aggs[a]
            isf = fn == "avg" or (fn != "count" and ctype[col] in ("f32", "f64"))
            return Pred(a, OPS[op], int(const) if not isf else 0, float(const))
        self.having = (Pred * max(1, len(hv)))(*[hpred(a, op, v) for a, op, v in hv])
        self.op = Operator(len(where), self.where, len(proj), self.proj, len(aggs), self.aggs,
                           len(gb), self.keys, len(hv), self.having)
        self.nkeys, self.aggs_spec = len(gb), list(aggs)
        self.key_dtypes = [np.int32 if ctype[c] == "i32" else np.int64 for c, _, _ in gb]
        self.agg_dtypes = []
        for fn, col in aggs:
            if fn == "count":
                self.agg_dtypes.append(np.int64)
            elif fn == "avg" or ctype[col] in ("f32", "f64"):
                self.agg_dtypes.append(np.float64)
            else:
                self.agg_dtypes.append(np.int64)


class Slice:
    """One polled result slice copied into numpy arrays (host mode)."""

    def __init__(self, task_id, first_window, nwindows, hdr, keys, vals, tuples):
        self.task_id, self.first_window, self.nwindows = task_id, first_window, nwindows
        self.hdr, self.keys, self.vals, self.tuples = hdr, keys, vals, tuples


class Query:
    """One windowed query on one GPU (wraps saber_query)."""

    def __init__(self, spec, device=None, task_bytes=64 << 20, result_mode=RESULTS_HOST, result_bytes=0,
                 hash_capacity=0, max_panes=0, base_index=0, first_window=0, emit_on_finish=True,
                 result_slots=8, pipeline_depth=3, profile=False):
        self.L = lib()
        self.m = _Marshalled(spec)
        self.spec = spec
        self.tuple_bytes = spec["schema"]["tuple_bytes"]
        cfg = Config()
        cfg.device = -1 if device is None else int(device)
        cfg.task_bytes = int(task_bytes)
        cfg.pipeline_depth = int(pipeline_depth)
        cfg.result_mode = int(result_mode)
        cfg.result_bytes = int(result_bytes)
        cfg.hash_capacity = int(hash_capacity)
        cfg.max_panes = int(max_panes)
        cfg.base_index = int(base_index)
        cfg.first_window = int(first_window)
        cfg.emit_on_finish = 1 if emit_on_finish else 0
        cfg.result_slots = int(result_slots)
        cfg.profile = 1 if profile else 0
        self.cfg = cfg
        h = C.c_void_p()
        _check(self.L.saber_query_create(C.byref(self.m.schema), C.byref(self.m.op), C.byref(self.m.window),
                                         C.byref(cfg), C.byref(h)))
        self.h = h
        self.result_mode = result_mode
        self._keep = []

    # -- ingest ---------------------------------------------------------------
    def submit(self, data):
        """Host tuples (bytes / numpy); blocks for staging, EAGAIN if result slots are full."""
        buf = np.ascontiguousarray(np.frombuffer(data, np.uint8) if isinstance(data, (bytes, bytearray))
                                   else np.asarray(data).view(np.uint8).reshape(-1))
        return self.L.saber_task_submit(self.h, buf.ctypes.data, buf.size)

    def submit_device(self, ptr, nbytes, stream=0):
        """Device tuples (a raw device pointer, e.g. torch tensor.data_ptr())."""
        return self.L.saber_task_submit_device(self.h, C.c_void_p(ptr), nbytes, C.c_void_p(stream))

    def register_host(self, arr):
        _check(self.L.saber_register_host(self.h, C.c_void_p(arr.ctypes.data), arr.nbytes), self.h)
        self._keep.append(arr)

    def finish(self, watermark=None):
        return self.L.saber_query_finish(self.h, -(1 << 63) if watermark is None else int(watermark))

    # -- results --------------------------------------------------------------
    def poll_raw(self, timeout_us=-1):
        r = Results()
        st = self.L.saber_results_poll(self.h, C.byref(r), int(timeout_us))
        return st, r

    def release(self, r):
        _check(self.L.saber_results_release(self.h, C.byref(r)), self.h)

    def poll(self, timeout_us=-1):
        """Next slice copied into numpy (host mode), or None if nothing is pending."""
        st, r = self.poll_raw(timeout_us)
        if st == EAGAIN:
            return None
        _check(st, self.h)
        try:
            if r.on_device:
                raise SaberError(EINVAL, "poll() copies host results; use poll_raw() in device mode")
            nw = r.nwindows
            hdr = np.zeros(nw, dtype=[("window_id", "<i8"), ("ts", "<i8"), ("row_offset", "<i8"),
                                      ("nrows", "<i4"), ("flags", "<i4")])
            if nw and r.hdr:
                C.memmove(hdr.ctypes.data, r.hdr, nw * 32)
            elif nw:   # σ/π (IStream) slices carry no per-window headers: ids only
                hdr["window_id"] = r.first_window + np.arange(nw)
                hdr["ts"] = -1
            keys, vals, tuples = [], [], b""
            if self.m.aggs_spec:
                for c in range(self.m.nkeys):
                    dt = self.m.key_dtypes[c]
                    a = np.empty(r.nrows, dtype=dt)
                    if r.nrows:
                        C.memmove(a.ctypes.data, r.cols[c], r.nrows * a.itemsize)
                    keys.append(a)
                for a_i, dt in enumerate(self.m.agg_dtypes):
                    a = np.empty(r.nrows, dtype=dt)
                    if r.nrows:
                        C.memmove(a.ctypes.data, r.cols[self.m.nkeys + a_i], r.nrows * 8)
                    vals.append(a)
            else:
                if r.ntuples:
                    tuples = C.string_at(r.tuples, r.ntuples * r.tuple_bytes)
            return Slice(r.task_id, r.first_window, nw, hdr, keys, vals, tuples)
        finally:
            self.release(r)

    def stats(self):
        s = Stats()
        _check(self.L.saber_query_stats(self.h, C.byref(s)), self.h)
        return {k: getattr(s, k) for k, _ in Stats._fields_}

    def sync(self):
        _check(self.L.saber_query_sync(self.h), self.h)

    def reset(self, base_index=0, first_window=0):
        """Restart on a new stream, keeping the plan and every buffer."""
        _check(self.L.saber_query_reset(self.h, int(base_index), int(first_window)), self.h)

    def record(self, stream=0):
        """Make CUDA stream `stream` wait for everything enqueued on this query."""
        _check(self.L.saber_query_record(self.h, C.c_void_p(stream)), self.h)

    def last_error(self):
        m = self.L.saber_last_error(self.h)
        return m.decode() if m else ""

    def close(self):
        if getattr(self, "h", None):
            self.L.saber_query_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- convenience: run a whole host stream through the query -----------------
    def run(self, data, chunk_bytes=None, watermark=None, finish=True):
        """Submit ``data`` in chunks (polling whenever result slots are full) and
        return all slices concatenated: dict(win_id, win_ts, win_nrows, keys, vals, tuples)."""
        buf = np.frombuffer(data, np.uint8) if isinstance(data, (bytes, bytearray)) else \
            np.asarray(data).view(np.uint8).reshape(-1)
        tb = self.tuple_bytes
        chunk = chunk_bytes or self.cfg.task_bytes
        chunk = min(chunk, self.cfg.task_bytes * max(1, self.cfg.result_slots - 1))
        chunk = max(tb, (chunk // tb) * tb)
        slices = []
        off = 0
        while off < buf.size:
            part = buf[off:off + chunk]
            st = self.submit(part)
            if st == EAGAIN:
                s = self.poll()
                if s is None:
                    _check(st, self.h)
                slices.append(s)
                continue
            _check(st, self.h)
            off += part.size
        if finish:
            while True:
                st = self.finish(watermark)
                if st == EAGAIN:
                    s = self.poll()
                    if s is None:
                        _check(st, self.h)
                    slices.append(s)
                    continue
                _check(st, self.h)
                break
        while True:
            s = self.poll()
            if s is None:
                break
            slices.append(s)
        return merge_slices(slices, self.m)


def merge_slices(slices, m):
    out = {"win_id": [], "win_ts": [], "win_nrows": [], "keys": [[] for _ in range(m.nkeys)],
           "vals": [[] for _ in m.aggs_spec], "tuples": []}
    for s in slices:
        out["win_id"].append(s.hdr["window_id"])
        out["win_ts"].append(s.hdr["ts"])
        out["win_nrows"].append(s.hdr["nrows"].astype(np.int64))
        for i, k in enumerate(s.keys):
            out["keys"][i].append(k)
        for i, v in enumerate(s.vals):
            out["vals"][i].append(v)
        out["tuples"].append(s.tuples)
    cat = lambda xs, dt: np.concatenate(xs) if xs else np.zeros(0, dt)  # noqa: E731
    res = {"win_id": cat(out["win_id"], np.int64), "win_ts": cat(out["win_ts"], np.int64),
           "win_nrows": cat(out["win_nrows"], np.int64),
           "keys": [cat(k, m.key_dtypes[i]) for i, k in enumerate(out["keys"])],
           "vals": [cat(v, m.agg_dtypes[i]) for i, v in enumerate(out["vals"])],
           "tuples": b"".join(out["tuples"])}
    return res


def partition_plan(spec, dev_ptr, begin, n):
    """(closed_windows, halo_first) for a contiguous partition held on the device."""
    m = _Marshalled(spec)
    c, h = C.c_int64(), C.c_int64()
    st = lib().saber_partition_plan(C.byref(m.schema), C.byref(m.window), C.c_void_p(dev_ptr), int(begin),
                                    int(n), C.byref(c), C.byref(h))
    _check(st)
    return c.value, h.value


class Join:
    """Windowed θ-join of two streams (wraps saber_join; include/saber.h).
    ``jspec``: schema1, schema2, window (count), theta [(col1, op, col2)],
    project1, project2 -- the dicts of saber_inputs.workloads.join_r."""

    def __init__(self, jspec, device=None, task_bytes=32 << 20, result_mode=RESULTS_HOST, result_bytes=0,
                 result_slots=4):
        self.L = lib()
        self.spec = jspec
        self.m1 = _Marshalled({"schema": jspec["schema1"], "window": jspec["window"]})
        self.m2 = _Marshalled({"schema": jspec["schema2"], "window": jspec["window"]})
        n1, n2 = self.m1.names, self.m2.names
        th = jspec.get("theta", [])
        self.theta = (JoinPred * max(1, len(th)))(*[JoinPred(n1.index(a), OPS[op], n2.index(b)) for a, op, b in th])
        self.p1 = (C.c_int32 * max(1, len(jspec["project1"])))(*[n1.index(c) for c in jspec["project1"]])
        self.p2 = (C.c_int32 * max(1, len(jspec["project2"])))(*[n2.index(c) for c in jspec["project2"]])
        self.op = JoinOp(len(th), self.theta, len(jspec["project1"]), self.p1, len(jspec["project2"]), self.p2)
        cfg = Config()
        cfg.device = -1 if device is None else int(device)
        cfg.task_bytes = int(task_bytes)
        cfg.result_mode = int(result_mode)
        cfg.result_bytes = int(result_bytes)
        cfg.result_slots = int(result_slots)
        self.cfg = cfg
        self.tb1, self.tb2 = jspec["schema1"]["tuple_bytes"], jspec["schema2"]["tuple_bytes"]
        h = C.c_void_p()
        st = self.L.saber_join_create(C.byref(self.m1.schema), C.byref(self.m2.schema), C.byref(self.op),
                                      C.byref(self.m1.window), C.byref(cfg), C.byref(h))
        if st != OK:
            raise SaberError(st, (self.L.saber_join_last_error(None) or b"").decode())
        self.h = h

    def last_error(self):
        m = self.L.saber_join_last_error(self.h)
        return m.decode() if m else ""

    def submit(self, d1, d2):
        b1 = np.ascontiguousarray(np.frombuffer(d1, np.uint8) if isinstance(d1, (bytes, bytearray)) else d1)
        b2 = np.ascontiguousarray(np.frombuffer(d2, np.uint8) if isinstance(d2, (bytes, bytearray)) else d2)
        n = b1.size // self.tb1
        assert b2.size // self.tb2 == n, "both batches of a task hold the same number of tuples"
        return self.L.saber_join_submit(self.h, C.c_void_p(b1.ctypes.data), C.c_void_p(b2.ctypes.data), n)

    def submit_device(self, ptr1, ptr2, ntuples, stream=0):
        return self.L.saber_join_submit_device(self.h, C.c_void_p(ptr1), C.c_void_p(ptr2), int(ntuples),
                                               C.c_void_p(stream))

    def poll_raw(self, timeout_us=-1):
        r = Results()
        return self.L.saber_join_poll(self.h, C.byref(r), int(timeout_us)), r

    def release(self, r):
        st = self.L.saber_join_release(self.h, C.byref(r))
        if st != OK:
            raise SaberError(st, self.last_error())

    def poll(self, timeout_us=-1):
        """Next slice copied into numpy (host mode): (headers, pair-row bytes), or None."""
        st, r = self.poll_raw(timeout_us)
        if st == EAGAIN:
            return None
        if st != OK:
            raise SaberError(st, self.last_error())
        try:
            hdr = np.zeros(r.nwindows, dtype=[("window_id", "<i8"), ("ts", "<i8"), ("row_offset", "<i8"),
                                              ("nrows", "<i4"), ("flags", "<i4")])
            if r.nwindows:
                C.memmove(hdr.ctypes.data, r.hdr, r.nwindows * 32)
            rows = C.string_at(r.tuples, r.ntuples * r.tuple_bytes) if r.ntuples else b""
            return hdr, rows
        finally:
            self.release(r)

    def run(self, d1, d2, batch_tuples):
        """Submit both streams in tasks of batch_tuples tuples; concatenated results."""
        n = min(len(d1) // self.tb1, len(d2) // self.tb2)
        hdrs, rows = [], []
        off = 0
        while off < n:
            k = min(batch_tuples, n - off)
            st = self.submit(d1[off * self.tb1:(off + k) * self.tb1], d2[off * self.tb2:(off + k) * self.tb2])
            if st == EAGAIN:
                h, r = self.poll()
                hdrs.append(h)
                rows.append(r)
                continue
            if st != OK:
                raise SaberError(st, self.last_error())
            off += k
        while (x := self.poll()) is not None:
            hdrs.append(x[0])
            rows.append(x[1])
        h = np.concatenate(hdrs) if hdrs else np.zeros(0, dtype=[("window_id", "<i8"), ("ts", "<i8"),
                                                                 ("row_offset", "<i8"), ("nrows", "<i4"),
                                                                 ("flags", "<i4")])
        return {"win_id": h["window_id"].astype(np.int64), "win_ts": h["ts"].astype(np.int64),
                "win_nrows": h["nrows"].astype(np.int64), "tuples": b"".join(rows)}

    def close(self):
        if getattr(self, "h", None):
            self.L.saber_join_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
