"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(device-resident stream from the device generator, the bench's task size φ,
RESULTS_DEVICE), on sampled windows the oracle evaluates one by one.

The oracle's input for a sampled window is generated on the host by the seeded
generator (saber_inputs.gen, byte-identical to the device twin -- a GPU test),
never copied from the CUDA path.  Samples include the first and last closed
window and windows straddling task boundaries (fragments assembled across
tasks, §4.3).  σ/π (C2) is checked by its IStream
property: the output is the projection of every selected, covered tuple, in
stream order (reading A9), at any size."""
import ctypes as C
import os

import numpy as np
import pytest

from parity import compare
from saber_inputs import gen, workloads

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


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
    import torch
    lib_gen = C.CDLL(os.path.join(ROOT, "saber_inputs", "libsaber_gen.so"))
    tb = spec["schema"]["tuple_bytes"]
    part = torch.empty(g["n"] * tb, dtype=torch.uint8, device="cuda")
    rc = lib_gen.saber_gen(gen.KIND_ID[g["kind"]], C.c_uint64(g["seed"]), C.c_int64(0), C.c_int64(g["n"]),
                           C.c_int64(g.get("rate", 1)), C.c_int64(g.get("groups", 64)),
                           C.c_void_p(part.data_ptr()), C.c_void_p(torch.cuda.current_stream().cuda_stream))
    assert rc == 0
    torch.cuda.synchronize()
    return part


def run_sampled(S, spec, g, task_bytes, sample):
    """Drive the whole stream through the C ABI like bench.py; keep the sampled
    windows' headers and rows (copied from the device result slots)."""
    import torch
    part = device_stream(spec, g)
    nk, na = len(spec.get("group_by", [])), len(spec["aggs"])
    q = S.Query(spec, task_bytes=task_bytes, result_mode=S.RESULTS_DEVICE, result_slots=8)
    want = set(int(j) for j in sample)
    got = {}

    def drain():
        st, r = q.poll_raw(-1)
        if st != 0:
            raise S.SaberError(st, q.last_error())
        try:
            for j in sorted(want):
                i = j - r.first_window
                if not 0 <= i < r.nwindows:
                    continue
                h = d2h(C.cast(r.hdr, C.c_void_p).value + 32 * i, 32).view(np.int64)
                wid, ts, off, nrows = int(h[0]), int(h[1]), int(h[2]), int(h[3] & 0xffffffff)
                assert wid == j
                keys = [d2h(r.cols[c] + off * r.col_bytes[c], nrows * r.col_bytes[c]).view(
                    np.int32 if r.col_bytes[c] == 4 else np.int64).astype(np.int64) for c in range(nk)]
                vals = [d2h(r.cols[nk + a] + off * 8, nrows * 8) for a in range(na)]
                got[j] = (ts, nrows, keys, vals)
        finally:
            q.release(r)

    stream = torch.cuda.current_stream().cuda_stream
    off, nbytes = 0, part.numel()
    while off < nbytes:
        nb = min(task_bytes, nbytes - off)
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
    return got


def oracle_window(oracle, spec, g, j):
    """The oracle on the tuples of window j only (host generator, same seed)."""
    w = spec["window"]
    rate = g.get("rate", 1)
    if w["kind"] == "count":
        i0, n = j * w["slide"], w["size"]
        data = gen.generate(g["kind"], n, g["seed"], i0=i0, rate=rate, groups=g.get("groups", 64))
        res = oracle.run(spec, data, windows=[0], nthreads=8)
        res["win_id"] = res["win_id"] + j
        return res
    t0 = w["origin"] + j * w["slide"]                      # ts = floor(i / rate) in the generator
    i0, n = t0 * rate, w["size"] * rate
    data = gen.generate(g["kind"], n, g["seed"], i0=i0, rate=rate, groups=g.get("groups", 64))
    return oracle.run(spec, data, windows=[j], watermark=t0 + w["size"], nthreads=8)


def as_result(spec, j, entry):
    ts, nrows, keys, vals = entry
    out = {"win_id": np.array([j], np.int64), "win_ts": np.array([ts], np.int64),
           "win_nrows": np.array([nrows], np.int64), "keys": keys, "vals": []}
    for a, (fn, col) in enumerate(spec["aggs"]):
        raw = vals[a]
        isf = fn == "avg" or (col is not None and dict((c[0], c[1]) for c in spec["schema"]["cols"])[col][0] == "f")
        out["vals"].append(raw.view(np.float64) if isf else raw.view(np.int64))
    return out


CASES = {
    # name: (workload, task bytes as bench.py times it, sampled windows)
    "C3_G64": (lambda: workloads.c3(groups=64), 4 << 30,
               [0, 1, 100000, 131040, 131041, 131056, 131071, 131072, 262112]),
    "C3_G65536": (lambda: workloads.c3(groups=65536), 256 << 20,
                  [0, 8160, 8161, 8190, 130000, 262112]),
    "C4_R64": (lambda: workloads.c4(rate=64), 4 << 30, [0, 1048500, 1048560, 1048575, 2097092]),
    "C5a": (lambda: workloads.c5a(), 4 << 30, [0, 29168, 32767, 61936]),
    "C5b": (lambda: workloads.c5b(), 4 << 30, [0, 16000, 16383, 16384, 32468]),
}


@pytest.mark.parametrize("name", list(CASES))
def test_full_size_sampled_windows(saber, oracle_lib, name):
    mk, task_bytes, sample = CASES[name]
    spec, g = mk()
    got = run_sampled(saber, spec, g, task_bytes, sample)
    assert sorted(got) == sorted(sample), f"windows not emitted: {sorted(set(sample) - set(got))}"
    for j in sample:
        compare(spec, as_result(spec, j, got[j]), oracle_window(oracle_lib, spec, g, j))


def test_c2_full_size_istream_property(saber):
    """C2 at full size (2^25 tuples, φ as bench.py): the IStream output equals the
    projection (ts, a1, a2) of every tuple with a3 < sel·2^31 whose position is
    covered by a closed window, in stream order."""
    import torch
    spec, g = workloads.c2(sel=0.5)
    part = device_stream(spec, g)
    q = saber.Query(spec, task_bytes=4 << 30, result_mode=saber.RESULTS_DEVICE, result_slots=8)
    outs = []
    stream = torch.cuda.current_stream().cuda_stream
    assert q.submit_device(part.data_ptr(), part.numel(), stream) == 0
    assert q.finish() == 0
    while q.stats()["tasks_pending"] > 0:
        st, r = q.poll_raw(-1)
        assert st == 0
        outs.append(d2h(r.tuples, r.ntuples * r.tuple_bytes))
        q.release(r)
    q.close()
    got = np.concatenate(outs) if outs else np.zeros(0, np.uint8)
    sdt = np.dtype([("ts", "<i8"), ("a1", "<f4"), ("a2", "<i4"), ("a3", "<i4"), ("a4", "<i4"), ("a5", "<i4"),
                    ("a6", "<i4")])
    a = np.ascontiguousarray(gen.generate_array("syn", g["n"], g["seed"])).view(sdt).reshape(-1)
    w = spec["window"]
    covered = ((g["n"] - w["size"]) // w["slide"]) * w["slide"] + w["size"]   # last closed window's end
    thr = spec["where"][0][2]
    sel = a[:covered][a["a3"][:covered] < thr]
    exp = np.zeros(len(sel), dtype=[("ts", "<i8"), ("a1", "<f4"), ("a2", "<i4")])
    for c in ("ts", "a1", "a2"):
        exp[c] = sel[c]
    assert got.size == exp.nbytes, (got.size, exp.nbytes)
    assert np.array_equal(got, exp.view(np.uint8))
