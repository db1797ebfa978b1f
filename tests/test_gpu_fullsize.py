"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (device-resident stream from the device generator, the bench's task size
φ from ``workloads.bench_task_mb``, RESULTS_DEVICE, 8 result slots).

SURVEY.md §8(c) C6 scale plan:
* C3 G=64 (the bench's default line), C1 and C2 (every selectivity run here at
  1 GiB): EVERY window is compared -- result slices are streamed back as the
  query runs and the oracle evaluates the same windows on a thread pool;
* every other config: the first 2^22 tuples' windows, the windows straddling
  every task boundary (fragments assembled across tasks, §4.3
  L1059-1091; for time windows whose span covers thousands of straddlers, the
  first and last 32 of each boundary and every 64th in between), 1,024 windows
  drawn with seed 0x5AB3, and the last window.
  C5a and SG1 (14.7 M tuples per window) draw 256 random windows by default.
* ``SABER_FULLSIZE=all`` draws all 1,024 random windows everywhere and streams
  EVERY window of C3 at G = 256 .. 4096 and C4 at R = 64 / 4096 (half an hour
  of oracle time on 16 cores; run on the GPU box, logs under profiles/r02/).
  C3 at G = 16K / 64K (4.5e9 / 6.8e9 result rows, a std::map per window in the
  oracle) stays sampled.

The oracle's input bytes are the seeded generator's (saber_inputs): the device
twin fills HBM for the product, the stream is copied to the host for the
oracle, and a sample of those host bytes is re-generated with the numpy
generator and must be identical (so no oracle input comes from the CUDA path).
Each test prints how many windows and rows it compared."""
import ctypes as C
import os
import threading
from concurrent.futures import ThreadPoolExecutor

import numpy as np
import pytest

from parity import compare
from saber_inputs import gen, workloads

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
FULL_ALL = os.environ.get("SABER_FULLSIZE", "") == "all"
NCPU = len(os.sched_getaffinity(0))


@pytest.fixture(scope="module")
def saber():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_sigmod_koliousiswfwcp16_b200 import saber as S
    return S


def d2h(ptr, nbytes):
    from cuda.bindings import runtime as rt
    out = np.empty(nbytes, np.uint8)
    if nbytes:
        (err,) = rt.cudaMemcpy(out.ctypes.data, int(ptr), nbytes, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost)
        assert int(err) == 0, err
    return out


def device_stream(spec, g):
    """(device tensor, host copy) of the workload's stream; the host copy is
    spot-checked against the numpy generator."""
    import torch
    lib_gen = C.CDLL(os.path.join(ROOT, "saber_inputs", "libsaber_gen.so"))
    tb = spec["schema"]["tuple_bytes"]
    part = torch.empty(g["n"] * tb, dtype=torch.uint8, device="cuda")
    rc = lib_gen.saber_gen(gen.KIND_ID[g["kind"]], C.c_uint64(g["seed"]), C.c_int64(0), C.c_int64(g["n"]),
                           C.c_int64(g.get("rate", 1)), C.c_int64(g.get("groups", 64)),
                           C.c_void_p(part.data_ptr()), C.c_void_p(torch.cuda.current_stream().cuda_stream))
    assert rc == 0
    torch.cuda.synchronize()
    host = part.cpu().numpy()
    rng = np.random.default_rng(0x5AB3)
    for i0 in list(rng.integers(0, g["n"] - 4096, size=6)) + [0, g["n"] - 4096]:
        exp = gen.generate(g["kind"], 4096, g["seed"], i0=int(i0), rate=g.get("rate", 1), groups=g.get("groups", 64))
        assert host[int(i0) * tb:(int(i0) + 4096) * tb].tobytes() == exp, "device generator differs from numpy"
    return part, host


def oracle_windows(oracle, spec, g, host, ids):
    """The oracle over windows ``ids`` (sorted), evaluated on runs of consecutive
    windows with the minimal slice of the host stream; results concatenated."""
    w = spec["window"]
    tb = spec["schema"]["tuple_bytes"]
    rate = g.get("rate", 1)
    n = host.size // tb
    ids = np.asarray(sorted(ids), np.int64)
    runs = np.split(ids, np.nonzero(np.diff(ids) != 1)[0] + 1) if ids.size else []
    parts = []

    def one(run):
        j0, j1 = int(run[0]), int(run[-1]) + 1
        if w["kind"] == "count":
            # IStream window j emits W_j \ W_{j-1}: start the slice at window j0-1
            # (position-relative window 0 would have no predecessor) and drop it
            k0 = 1 if (not spec.get("aggs") and j0 > 0) else 0
            a, b = (j0 - k0) * w["slide"], (j1 - 1) * w["slide"] + w["size"]
            r = oracle.run(spec, host[a * tb:b * tb], windows=list(range(k0, j1 - j0 + k0)),
                           nthreads=max(1, NCPU // 4))
            r["win_id"] = r["win_id"] + j0 - k0
            return r
        t_lo, t_hi = w["origin"] + j0 * w["slide"], w["origin"] + (j1 - 1) * w["slide"] + w["size"]
        a, b = min(n, t_lo * rate), min(n, t_hi * rate)        # ts = floor(i / rate) in the generator
        return oracle.run(spec, host[a * tb:b * tb], windows=list(range(j0, j1)), watermark=t_hi,
                          nthreads=max(1, NCPU // 4))
    # split long runs so the pool stays busy
    chunks = []
    for run in runs:
        step = 4096 if w["kind"] == "count" else 64
        chunks += [run[i:i + step] for i in range(0, len(run), step)]
    with ThreadPoolExecutor(max_workers=4) as ex:
        parts = list(ex.map(one, chunks))
    return concat_results(spec, parts)


def concat_results(spec, parts):
    na = len(spec.get("aggs", []))
    nk = len(spec.get("group_by", []))
    if not parts:
        return {"win_id": np.zeros(0, np.int64), "win_ts": np.zeros(0, np.int64), "win_nrows": np.zeros(0, np.int64),
                "keys": np.zeros((0, nk), np.int64), "vals": [np.zeros(0) for _ in range(na)], "tuples": b""}
    return {"win_id": np.concatenate([p["win_id"] for p in parts]),
            "win_ts": np.concatenate([p["win_ts"] for p in parts]),
            "win_nrows": np.concatenate([p["win_nrows"] for p in parts]),
            "keys": np.concatenate([p["keys"] for p in parts]) if nk else np.zeros((sum(len(p["keys"]) for p in parts), 0), np.int64),
            "vals": [np.concatenate([p["vals"][a] for p in parts]) for a in range(na)],
            "tuples": b"".join(p["tuples"] for p in parts)}


def slice_windows(spec, r, want=None):
    """Headers and rows of a polled device slice (all windows, or the sorted
    window ids in ``want`` that fall into it) as a result dict."""
    nk, na = len(spec.get("group_by", [])), len(spec.get("aggs", []))
    nw = int(r.nwindows)
    hdr = d2h(C.cast(r.hdr, C.c_void_p).value, nw * 32).view(np.int64).reshape(nw, 4) if nw else np.zeros((0, 4), np.int64)
    idx = np.arange(nw) if want is None else (np.asarray(want, np.int64) - int(r.first_window))
    idx = idx[(idx >= 0) & (idx < nw)]
    h = hdr[idx]
    wid, ts, off = h[:, 0], h[:, 1], h[:, 2]
    nrows = (h[:, 3] & 0xffffffff).astype(np.int64)
    out = {"win_id": wid.copy(), "win_ts": ts.copy(), "win_nrows": nrows, "tuples": b""}
    if na == 0:                                       # σ/π: the projected tuples of these windows
        tbo = r.tuple_bytes
        if want is None:
            out["tuples"] = d2h(r.tuples, r.ntuples * tbo).tobytes()
        else:
            out["tuples"] = b"".join(d2h(r.tuples + int(o) * tbo, int(c) * tbo).tobytes() for o, c in zip(off, nrows))
        return out
    keys, vals = [[] for _ in range(nk)], [[] for _ in range(na)]
    ctype = {c[0]: c[1] for c in spec["schema"]["cols"]}
    isf = [fn == "avg" or (fn != "count" and ctype[col][0] == "f") for fn, col in spec["aggs"]]
    if want is None and nw:
        o0, o1 = int(off[0]), int(off[-1] + nrows[-1])
        segs = [(o0, o1 - o0)]
    else:
        segs = [(int(o), int(c)) for o, c in zip(off, nrows)]
    for o, cnt in segs:
        for c in range(nk):
            b = r.col_bytes[c]
            keys[c].append(d2h(r.cols[c] + o * b, cnt * b).view(np.int32 if b == 4 else np.int64).astype(np.int64))
        for a in range(na):
            v = d2h(r.cols[nk + a] + o * 8, cnt * 8)
            vals[a].append(v.view(np.float64) if isf[a] else v.view(np.int64))
    out["keys"] = [np.concatenate(k) if k else np.zeros(0, np.int64) for k in keys]
    out["vals"] = [np.concatenate(v) if v else np.zeros(0) for v in vals]
    return out


def merge_got(spec, parts):
    nk, na = len(spec.get("group_by", [])), len(spec.get("aggs", []))
    out = {"win_id": np.concatenate([p["win_id"] for p in parts]) if parts else np.zeros(0, np.int64),
           "win_ts": np.concatenate([p["win_ts"] for p in parts]) if parts else np.zeros(0, np.int64),
           "win_nrows": np.concatenate([p["win_nrows"] for p in parts]) if parts else np.zeros(0, np.int64),
           "tuples": b"".join(p["tuples"] for p in parts)}
    if na:
        out["keys"] = [np.concatenate([p["keys"][c] for p in parts]) for c in range(nk)]
        out["vals"] = [np.concatenate([p["vals"][a] for p in parts]) for a in range(na)]
    return out


def run_stream(S, oracle, spec, g, task_bytes, sample=None, full=False):
    """Drive the whole stream through the C ABI like bench.py.  ``full``: compare
    every window of every slice against the oracle as slices arrive (the oracle
    runs on a worker thread while the GPU continues); else compare the windows in
    ``sample`` (a callable n_windows -> ids, or an id list).  Returns
    (windows compared, rows compared, total windows)."""
    import torch
    part, host = device_stream(spec, g)
    q = S.Query(spec, task_bytes=task_bytes, result_mode=S.RESULTS_DEVICE, result_slots=8)
    stats = {"windows": 0, "rows": 0, "total": 0}
    pending = []
    lock = threading.Lock()
    pool = ThreadPoolExecutor(max_workers=1)
    want = None
    got_sample = []
    w = spec["window"]
    tb = spec["schema"]["tuple_bytes"]
    if not full:
        if w["kind"] == "count":
            nwin = (g["n"] - w["size"]) // w["slide"] + 1
        else:
            tl = (g["n"] - 1) // g.get("rate", 1)
            nwin = (tl + 1 - w["origin"] - w["size"]) // w["slide"] + 1
        want = sorted(set(int(j) for j in (sample(nwin, q) if callable(sample) else sample) if 0 <= j < nwin))

    def check(got):
        exp = oracle_windows(oracle, spec, g, host, got["win_id"])
        compare(spec, got, exp)
        with lock:
            stats["windows"] += len(got["win_id"])
            stats["rows"] += int(got["win_nrows"].sum())

    def drain():
        st, r = q.poll_raw(-1)
        if st != 0:
            raise S.SaberError(st, q.last_error())
        try:
            stats["total"] += int(r.nwindows)
            if full:
                got = slice_windows(spec, r)
                pending.append(pool.submit(check, got))
                if len(pending) > 2:
                    pending.pop(0).result()
            else:
                got_sample.append(slice_windows(spec, r, want))
        finally:
            q.release(r)

    stream = torch.cuda.current_stream().cuda_stream
    off, nbytes = 0, part.numel()
    eff = q.stats()["task_tuples"] * tb             # effective φ (the dispatcher may cut smaller tasks)
    while off < nbytes:
        nb = min(eff, nbytes - off)
        st = q.submit_device(part.data_ptr() + off, nb, stream)
        if st == S.EAGAIN:
            drain()
            continue
        assert st == 0, q.last_error()
        off += nb
    while (st := q.finish()) == S.EAGAIN:
        drain()
    assert st == 0, q.last_error()
    while q.stats()["tasks_pending"] > 0:
        drain()
    q.close()
    del part
    torch.cuda.empty_cache()
    for f in pending:
        f.result()
    pool.shutdown()
    if not full:
        got = merge_got(spec, got_sample)
        assert list(got["win_id"]) == want, "sampled windows not all emitted"
        check(got)
    return stats["windows"], stats["rows"], stats["total"]


def c6_sample(spec, g, task_bytes, nrand=1024):
    """first 2^22 tuples' windows, task-boundary straddlers,
    ``nrand`` (1,024) seeded windows (0x5AB3), the last window."""
    w = spec["window"]
    tb = spec["schema"]["tuple_bytes"]
    rate = g.get("rate", 1)
    tt = task_bytes // tb

    def ids(nwin, q):
        s, l = w["size"], w["slide"]
        tt = q.stats()["task_tuples"]                  # effective φ (the dispatcher may cut smaller tasks)
        out = set()
        if w["kind"] == "count":
            out.update(range(0, max(0, ((1 << 22) - s) // l + 1)))
            for b in range(tt, g["n"], tt):              # windows with start < b <= end
                lo, hi = max(0, (b - s) // l), min(nwin, (b - 1) // l + 1)
                strad = list(range(lo, hi))
                out.update(strad if len(strad) <= 96 else strad[:32] + strad[-32:] + strad[32:-32:64])
        else:
            T0 = w["origin"]
            last_t = ((1 << 22) - 1) // rate
            out.update(range(0, max(0, (last_t + 1 - T0 - s) // l + 1)))
            for b in range(tt, g["n"], tt):
                tb_ = b // rate                          # τ at the cut
                lo, hi = max(0, (tb_ - T0 - s) // l), min(nwin, (tb_ - T0) // l + 1)
                strad = list(range(lo, hi))
                out.update(strad if len(strad) <= 96 else strad[:32] + strad[-32:] + strad[32:-32:64])
        rng = np.random.default_rng(0x5AB3)
        out.update(int(x) for x in rng.integers(0, nwin, size=nrand))
        out.add(nwin - 1)
        return out
    return ids


FULL = {
    # name: (workload, compare every window)
    "C3_G64": (lambda: workloads.c3(groups=64), "C3", 64, True),
    "C1_sum": (lambda: workloads.c1("sum"), "C1", 64, True),
    "C1_max": (lambda: workloads.c1("max"), "C1", 64, True),
    "C2_sel0.5": (lambda: workloads.c2(sel=0.5, n=1 << 25), "C2", 64, True),
    "C2_sel0.01": (lambda: workloads.c2(sel=0.01, n=1 << 25), "C2", 64, True),
    "C3_G256": (lambda: workloads.c3(groups=256), "C3", 256, False),
    "C3_G1024": (lambda: workloads.c3(groups=1024), "C3", 1024, False),
    "C3_G4096": (lambda: workloads.c3(groups=4096), "C3", 4096, False),
    "C3_G16384": (lambda: workloads.c3(groups=16384), "C3", 16384, False),
    "C3_G65536": (lambda: workloads.c3(groups=65536), "C3", 65536, False),
    # φ = 4 GiB requested: one task would close 131K windows x up to 32,768 rows, more
    # than a 4 GiB result slot; the dispatcher cuts smaller tasks instead of failing
    "C3_G65536_phi4G": (lambda: workloads.c3(groups=65536), "C3", -4096, False),
    "C4_R64": (lambda: workloads.c4(rate=64), "C4", 64, False),
    "C4_R4096": (lambda: workloads.c4(rate=4096), "C4", 64, False),
    "C5a": (lambda: workloads.c5a(), "C5a", 64, False),
    "C5b": (lambda: workloads.c5b(), "C5b", 64, False),
    "SG1": (lambda: workloads.sg1(), "SG1", 64, False),
}
EVERY_WINDOW_WHEN_ALL = {"C3_G256", "C3_G1024", "C3_G4096", "C4_R64", "C4_R4096"}


@pytest.mark.parametrize("name", list(FULL))
def test_full_size(saber, oracle_lib, name):
    mk, cfg, groups, full = FULL[name]
    spec, g = mk()
    task_bytes = (workloads.bench_task_mb(cfg, groups) if groups > 0 else -groups) << 20
    groups = abs(groups)
    full = full or (FULL_ALL and name in EVERY_WINDOW_WHEN_ALL)
    # C5a / SG1 windows span 3,600 s x 4,096 tuples/s = 14.7 M tuples each: the
    # default run draws 256 random windows (~2 min of oracle time), SABER_FULLSIZE=all 1,024
    nrand = 256 if (name in ("C5a", "SG1") and not FULL_ALL) else 1024
    sample = None if full else c6_sample(spec, g, task_bytes, nrand)
    nw, nr, total = run_stream(saber, oracle_lib, spec, g, task_bytes, sample=sample, full=full)
    print(f"\n[fullsize] {name}: {'every window' if full else 'C6 sample'}: {nw} of {total} windows, "
          f"{nr} rows compared (phi = {task_bytes >> 20} MiB)")
    assert nw > 0
    if full:
        assert nw == total
