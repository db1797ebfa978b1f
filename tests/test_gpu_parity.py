"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by
element on the same seeded inputs (run with -m gpu on a B200)."""
import numpy as np
import pytest

from parity import compare
from saber_inputs import gen, workloads
from tiny import TINY, golden, spec as tspec, stream

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def saber():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_sigmod_koliousiswfwcp16_b200 import saber as S
    return S


def run_product(S, spec, data, task_bytes=1 << 20, watermark=None, chunk_bytes=None, **kw):
    q = S.Query(spec, task_bytes=task_bytes, **kw)
    try:
        return q.run(data, chunk_bytes=chunk_bytes, watermark=watermark)
    finally:
        q.close()


def check(S, oracle_lib, spec, data, watermark=None, **kw):
    exp = oracle_lib.run(spec, data, watermark=watermark, nthreads=8)
    got = run_product(S, spec, data, watermark=watermark, **kw)
    compare(spec, got, exp)
    return got, exp


# ------------------------------------------------------------------ goldens --
@pytest.mark.parametrize("gid", ["G1", "G2", "G3"])
@pytest.mark.parametrize("task_tuples", [1, 3, 5, 64])
def test_golden_count(saber, oracle_lib, gid, task_tuples):
    g = golden(gid)
    sp = tspec(g["window"], aggs=[("sum", "v"), ("count", None), ("min", "v"), ("max", "x")])
    got, _ = check(saber, oracle_lib, sp, stream(v=g["tuples_v"], x=np.arange(10) / 4.0),
                   task_bytes=32 * task_tuples)
    assert list(got["vals"][0]) == g["expect_sum"]


def test_golden_fragment_classes(saber):
    """Fig. 2 prose (L508-517): per-task window-fragment classes for 5-tuple tasks."""
    for gid in ("G1", "G2"):
        g = golden(gid)
        sp = tspec(g["window"], aggs=[("sum", "v")])
        q = saber.Query(sp, task_bytes=32 * g["task_tuples"])
        d = stream(v=g["tuples_v"])
        for t, cls in enumerate(g["expect_task_classes"]):
            assert q.submit(d[t * 160:(t + 1) * 160]) == 0
            st = q.stats()
            assert (st["last_complete"], st["last_opening"], st["last_closing"], st["last_pending"]) == \
                (len(cls["complete"]), len(cls["opening"]), len(cls["closing"]), len(cls["pending"])), (gid, t)
        q.close()


@pytest.mark.parametrize("task_tuples", [1, 2, 4, 10])
def test_golden_time(saber, oracle_lib, task_tuples):
    g = golden("G4")
    d = stream(v=g["tuples_v"], tau=g["tau"])
    for w in ({"kind": "time", "size": 3, "slide": 1}, {"kind": "time", "size": 1, "slide": 1},
              {"kind": "time", "size": 2, "slide": 2}):
        sp = tspec(w, aggs=[("count", None), ("sum", "v")])
        check(saber, oracle_lib, sp, d, task_bytes=32 * task_tuples)


def test_golden_groupby_having_istream(saber, oracle_lib):
    g6 = golden("G6")
    d = stream(x=g6["x"], k=g6["key"])
    for dom in (0, 3):
        sp = tspec(g6["window"], aggs=[("sum", "x"), ("count", None), ("avg", "x")], group_by=[("k", 1, dom)])
        check(saber, oracle_lib, sp, d, task_bytes=64)
        sp = tspec(g6["window"], aggs=[("avg", "x")], group_by=[("k", 1, dom)], having=[(0, "<", 1.0)])
        check(saber, oracle_lib, sp, d, task_bytes=96)
    g7 = golden("G7")
    sp = tspec(g7["window"], where=[("o", "==", 1)], project=["v"])
    got, _ = check(saber, oracle_lib, sp, stream(v=g7["tuples_v"]), task_bytes=64)
    assert list(np.frombuffer(got["tuples"], np.int32)) == g7["expect_v"]


# -------------------------------------------------------------- configs -------
@pytest.mark.parametrize("fn", ["sum", "count", "avg", "min", "max"])
def test_c1_full_size(saber, oracle_lib, fn):
    """configs[0] at its full size (1M tuples), one task and many tasks."""
    spec, g = workloads.c1(fn)
    data = gen.generate("syn", g["n"], g["seed"], rate=g["rate"], groups=g["groups"])
    check(saber, oracle_lib, spec, data, task_bytes=32 << 20)
    check(saber, oracle_lib, spec, data, task_bytes=(1 << 20) + 4096)


@pytest.mark.parametrize("sel", [0.0, 0.01, 0.5, 1.0])
def test_c2_select_project(saber, oracle_lib, sel):
    spec, g = workloads.c2(sel=sel, npred=4 if sel == 0.5 else 1)
    n = 1 << 20
    data = gen.generate("syn", n, g["seed"], rate=1)
    check(saber, oracle_lib, spec, data, task_bytes=(4 << 20) + 32 * 77)


@pytest.mark.parametrize("groups,dom", [(64, True), (64, False), (200, True), (300, True), (1024, True), (4096, True), (16384, True), (65536, False)])
def test_c3_groupby(saber, oracle_lib, groups, dom):
    spec, g = workloads.c3(groups=groups, declare_domain=dom)
    n = 1 << 19
    data = gen.generate("syn", n, g["seed"], rate=1, groups=groups)
    check(saber, oracle_lib, spec, data, task_bytes=(4 << 20))


# bucket mode (k_bucket.cu): count windows, one int32 key with a large declared
# domain; ragged task sizes, several key slabs, σ, 0/1/2 accumulator fields
@pytest.mark.parametrize("case", ["g64k_ragged", "g20000_sigma", "g100000_tumbling", "cm_two_fields", "count_only"])
def test_bucket_mode(saber, oracle_lib, case):
    if case == "g64k_ragged":
        spec, g = workloads.c3(groups=65536)
        data = gen.generate("syn", 1 << 19, g["seed"], rate=1, groups=65536)
        tb = (4 << 20) + 32 * 77
    elif case == "g20000_sigma":
        spec, _ = workloads.c3(groups=20000)
        spec["window"] = workloads.count_window(4096, 512)
        spec["aggs"] = [("count", None), ("sum", "a1"), ("avg", "a1")]
        spec["where"] = [("a3", "<", int(0.7 * 2 ** 31))]
        data = gen.generate("syn", 200000, 11, rate=1, groups=20000)
        tb = (1 << 20) + 32 * 5
    elif case == "g100000_tumbling":
        spec, _ = workloads.c3(groups=100000)
        spec["window"] = workloads.count_window(2048, 2048)
        data = gen.generate("syn", 300000, 12, rate=1, groups=100000)
        tb = 777 * 32
    elif case == "cm_two_fields":
        spec, _ = workloads.c4(gcat=32768)
        spec["window"] = workloads.count_window(3000, 1000)
        spec["aggs"] = [("sum", "cpu"), ("avg", "ram"), ("count", None)]
        data = gen.generate("cm", 150000, 13, rate=64, groups=32768)
        tb = (2 << 20) + 64 * 3
    else:
        spec, _ = workloads.c3(groups=50000)
        spec["window"] = workloads.count_window(1500, 300)
        spec["aggs"] = [("count", None)]
        data = gen.generate("syn", 100000, 14, rate=1, groups=50000)
        tb = 1 << 20
    check(saber, oracle_lib, spec, data, task_bytes=tb)


@pytest.mark.parametrize("rate", [64, 4096])
def test_c4_cm1(saber, oracle_lib, rate):
    spec, g = workloads.c4(rate=rate)
    n = 1 << 18
    data = gen.generate("cm", n, g["seed"], rate=rate, groups=g["groups"])
    check(saber, oracle_lib, spec, data, task_bytes=(2 << 20))


@pytest.mark.parametrize("rate", [128, 4096])
def test_c4_table_layout_switch(saber, oracle_lib, rate):
    """Time windows with GROUP BY start with warp tables and switch to lane-private
    tables once polled tasks (>= 1M tuples) show long panes: results must not change."""
    spec, g = workloads.c4(rate=rate)
    n = 1 << 22
    data = gen.generate("cm", n, g["seed"], rate=rate, groups=g["groups"])
    tb = len(data) // n
    check(saber, oracle_lib, spec, data, task_bytes=tb * (1 << 20), result_slots=2)


def test_c5a_sg2_and_sg1(saber, oracle_lib):
    for spec, g in (workloads.c5a(), workloads.sg1()):
        spec["window"]["size"] = 60          # shorter window so the oracle stays fast
        n = 1 << 19
        data = gen.generate("sg", n, g["seed"], rate=1024)
        check(saber, oracle_lib, spec, data, task_bytes=(2 << 20))


def test_c5b_lrb3(saber, oracle_lib):
    spec, g = workloads.c5b()
    spec["window"]["size"] = 30
    n = 1 << 19
    data = gen.generate("lrb", n, g["seed"], rate=2048)
    check(saber, oracle_lib, spec, data, task_bytes=(2 << 20))


def test_cm2_int64_key_hash(saber, oracle_lib):
    spec, g = workloads.cm2(rate=64)
    n = 1 << 17
    data = gen.generate("cm", n, g["seed"], rate=64, groups=4)
    check(saber, oracle_lib, spec, data, task_bytes=(1 << 20))


# ----------------------------------------------------- random small streams --
def _random_case(rng):
    n = int(rng.integers(0, 3000))
    s = int(rng.integers(1, 200))
    l = int(rng.integers(1, s + 1))
    kind = "count" if rng.random() < 0.5 else "time"
    tau = np.cumsum(rng.choice([0, 0, 1, 1, 2, 5], size=n)) if kind == "time" else np.arange(n)
    v = rng.integers(-1000, 1000, size=n)
    x = rng.integers(0, 1 << 12, size=n) / 64.0
    k = rng.integers(0, int(rng.choice([1, 3, 17, 300])), size=n)
    w = {"kind": kind, "size": s, "slide": l, "origin": int(rng.integers(0, 3)) if kind == "time" else 0}
    where = [("v", "<", int(rng.integers(-500, 1000)))] if rng.random() < 0.4 else []
    if rng.random() < 0.2:
        sp = tspec(w, where=where, project=list(rng.choice(["ts", "v", "x", "k", "m"], size=int(rng.integers(1, 4)))))
    else:
        fns = ["sum", "count", "avg", "min", "max"]
        aggs = []
        for _ in range(int(rng.integers(1, 4))):
            fn = str(rng.choice(fns))
            aggs.append((fn, None) if fn == "count" else (fn, str(rng.choice(["v", "x"]))))
        gb = []
        r = rng.random()
        if r < 0.35:
            gb = [("k", 1, 300 if rng.random() < 0.5 else 0)]
        elif r < 0.5:
            gb = [("k", 1, 0), ("v", 7, 0)]
        elif r < 0.6:
            gb = [("k", 1, 300), ("o", 1, 2)]
        having = [(0, ">=", 0.0)] if rng.random() < 0.2 else []
        sp = tspec(w, where=where, aggs=aggs, group_by=gb, having=having)
    return sp, stream(v=v, tau=tau, x=x, k=k, n=n)


@pytest.mark.parametrize("seed", range(6))
def test_random_streams(saber, oracle_lib, seed):
    rng = np.random.default_rng(77 + seed)
    for _ in range(12):
        sp, d = _random_case(rng)
        tt = int(rng.choice([1, 7, 100, 1000, 5000]))
        wm = None
        if sp["window"]["kind"] == "time" and rng.random() < 0.3 and len(d):
            wm = int(np.frombuffer(d, np.int64).reshape(-1, 4)[-1, 0] + rng.integers(0, 50))
        chunk = int(rng.choice([32, 32 * 13, 32 * 1000])) if rng.random() < 0.5 else None
        check(saber, oracle_lib, sp, d, watermark=wm, task_bytes=32 * tt, chunk_bytes=chunk)


# --------------------------------------------------------------- invariants --
def test_task_size_invariance(saber, oracle_lib):
    """A22 / Fig. 13: results do not depend on the task size φ (ints bit-exact)."""
    spec, g = workloads.c3(groups=256)
    spec["aggs"] = [("count", None), ("sum", "a3"), ("max", "a1"), ("avg", "a1")]
    spec["window"] = workloads.count_window(4096, 512)
    data = gen.generate("syn", 1 << 18, 9, groups=256)
    exp = oracle_lib.run(spec, data, nthreads=8)
    for tb in (32 * 999, 1 << 20, 3 << 20, 8 << 20):
        compare(spec, run_product(saber, spec, data, task_bytes=tb), exp)


def test_device_submit_matches_host(saber, oracle_lib):
    import torch
    spec, g = workloads.c4(rate=64)
    n = 1 << 17
    data = gen.generate("cm", n, g["seed"], rate=64, groups=4)
    exp = oracle_lib.run(spec, data, nthreads=8)
    dev = torch.from_numpy(np.frombuffer(data, np.uint8).copy()).cuda()
    q = saber.Query(spec, task_bytes=1 << 20)
    slices = []
    off, tb = 0, 1 << 20
    while off < dev.numel():
        nb = min(tb * 2, dev.numel() - off)
        st = q.submit_device(dev.data_ptr() + off, nb, torch.cuda.current_stream().cuda_stream)
        if st == saber.EAGAIN:
            slices.append(q.poll())
            continue
        assert st == 0, q.last_error()
        off += nb
    while (st := q.finish()) == saber.EAGAIN:
        slices.append(q.poll())
    assert st == 0, q.last_error()
    while (s := q.poll()) is not None:
        slices.append(s)
    compare(spec, saber.merge_slices(slices, q.m), exp)
    q.close()


# ------------------------------------------------------------------- errors --
def test_errors_are_sticky(saber):
    sp = tspec({"kind": "time", "size": 2, "slide": 1}, aggs=[("count", None)])
    q = saber.Query(sp, task_bytes=32 * 4)
    q.submit(stream(tau=[0, 1, 2, 1, 3, 4, 5, 6]))
    q.finish()
    with pytest.raises(saber.SaberError) as e:
        while q.poll() is not None:
            pass
    assert e.value.status == saber.EORDER
    q.close()
    sp = tspec({"kind": "count", "size": 2, "slide": 1}, aggs=[("count", None)], group_by=[("k", 1, 2)])
    q = saber.Query(sp, task_bytes=32 * 4)
    q.submit(stream(k=[0, 1, 5, 1]))
    q.finish()
    with pytest.raises(saber.SaberError) as e:
        while q.poll() is not None:
            pass
    assert e.value.status == saber.EKEY
    q.close()


def test_invalid_queries_rejected(saber):
    with pytest.raises(saber.SaberError) as e:
        saber.Query(tspec({"kind": "count", "size": 2, "slide": 3}, aggs=[("count", None)]))
    assert e.value.status == saber.EINVAL
    with pytest.raises(saber.SaberError):
        saber.Query(tspec({"kind": "count", "size": 2, "slide": 1}, aggs=[("sum", "x")], group_by=[("x", 1, 0)]))


def test_device_generator_matches_numpy(saber):
    import ctypes as C
    import os
    import torch
    L = C.CDLL(os.path.join(os.path.dirname(gen.__file__), "libsaber_gen.so"))
    for kind, tb in (("syn", 32), ("cm", 64), ("sg", 32), ("lrb", 32)):
        n, i0 = 5000, 123456789
        buf = torch.empty(n * tb, dtype=torch.uint8, device="cuda")
        L.saber_gen(gen.KIND_ID[kind], C.c_uint64(7), C.c_int64(i0), C.c_int64(n), C.c_int64(3), C.c_int64(64),
                    C.c_void_p(buf.data_ptr()), None)
        torch.cuda.synchronize()
        assert buf.cpu().numpy().tobytes() == gen.generate(kind, n, 7, i0=i0, rate=3, groups=64), kind


# ------------------------------------------------------- task partitioning ---
@pytest.mark.parametrize("cfg", ["count", "time", "istream_time"])
@pytest.mark.parametrize("parts", [2, 3])
def test_partitioned_queries_match_single_gpu(saber, oracle_lib, cfg, parts):
    """The multi-GPU plan, run as sequential partitions on one GPU: each partition
    gets its predecessor's halo (saber_partition_plan on the device), base_index
    and first_window, and only the last emits on finish."""
    import torch
    if cfg == "count":
        spec, g = workloads.c3(groups=64)
        spec["window"] = workloads.count_window(4096, 512)
        n = 1 << 17
    elif cfg == "time":
        spec, g = workloads.c4(rate=97)
        n = 1 << 17
    else:
        spec, g = workloads.c2(sel=0.3)
        spec["window"] = workloads.time_window(50, 7)
        g = dict(g, rate=13)
        n = 1 << 16
    data = gen.generate(g["kind"], n, g["seed"], rate=g["rate"], groups=g.get("groups", 64))
    tb = spec["schema"]["tuple_bytes"]
    dev = torch.from_numpy(np.frombuffer(data, np.uint8).copy()).cuda()
    exp = oracle_lib.run(spec, data, nthreads=8)
    bounds = [(r * n // parts, (r + 1) * n // parts) for r in range(parts)]
    slices, first_window, base_index = [], 0, 0
    for r, (b, e) in enumerate(bounds):
        q = saber.Query(spec, task_bytes=(1 << 20) + tb * 11, base_index=base_index, first_window=first_window,
                        emit_on_finish=(r == parts - 1))
        got = q.run(np.frombuffer(data, np.uint8)[base_index * tb:e * tb])
        q.close()
        slices.append(got)
        if r < parts - 1:
            first_window, base_index = saber.partition_plan(spec, dev.data_ptr() + b * tb, b, e - b)
    merged = {"win_id": np.concatenate([s["win_id"] for s in slices]),
              "win_ts": np.concatenate([s["win_ts"] for s in slices]),
              "win_nrows": np.concatenate([s["win_nrows"] for s in slices]),
              "keys": [np.concatenate([s["keys"][i] for s in slices]) for i in range(len(slices[0]["keys"]))],
              "vals": [np.concatenate([s["vals"][i] for s in slices]) for i in range(len(slices[0]["vals"]))],
              "tuples": b"".join(s["tuples"] for s in slices)}
    compare(spec, merged, exp)


# ------------------------------------------------- overlapped window phase --
@pytest.mark.parametrize("case", ["c3_g64", "c3_minmax_ragged", "c4_time", "sg_long", "c1_tumbling"])
def test_overlap_window_phase(saber, oracle_lib, case, monkeypatch):
    """Plan::overlap (SABER_OVERLAP=1): the window phase of task i runs on a second
    stream on a State snapshot while task i+1 scans; results must equal the oracle
    (many small tasks, ragged sizes, fewer result slots than tasks)."""
    monkeypatch.setenv("SABER_OVERLAP", "1")
    if case == "c3_g64":
        spec, g = workloads.c3(groups=64)
        spec["window"] = workloads.count_window(4096, 1024)
        data = gen.generate("syn", 1 << 18, g["seed"], groups=64)
        tb = 1 << 20
    elif case == "c3_minmax_ragged":
        spec, g = workloads.c3(groups=32)
        spec["window"] = workloads.count_window(2048, 256)
        spec["aggs"] = [("min", "a1"), ("max", "a3"), ("count", None), ("sum", "a4")]
        data = gen.generate("syn", 300000, 21, groups=32)
        tb = 32 * 20011
    elif case == "c4_time":
        spec, g = workloads.c4(rate=64)
        data = gen.generate("cm", 1 << 18, g["seed"], rate=64, groups=g["groups"])
        tb = 64 * 7001
    elif case == "sg_long":
        spec, g = workloads.c5a()
        spec["window"]["size"] = 120
        data = gen.generate("sg", 1 << 19, g["seed"], rate=512)
        tb = 32 * 50000
    else:
        spec, g = workloads.c1()
        data = gen.generate("syn", 1 << 18, g["seed"])
        tb = 32 * 3000
    check(saber, oracle_lib, spec, data, task_bytes=tb, result_slots=3)


@pytest.mark.parametrize("seed", range(3))
def test_radix_keys_with_divisors(saber, oracle_lib, seed):
    """k_pane_agg fast path for several radix-packed int32 keys (Plan::fast_keys):
    key = (k, v / d) with C truncation (reading A17) -- negative v in (-d, 0) map to
    key 0 -- and sums/averages of the f32 column, count and time windows."""
    rng = np.random.default_rng(500 + seed)
    n = 20000
    d = int(rng.choice([3, 7, 5280 // 64]))
    v = rng.integers(-d + 1, 40 * d, size=n)
    x = rng.integers(0, 1 << 12, size=n) / 64.0
    k = rng.integers(0, 5, size=n)
    for kind in ("count", "time"):
        tau = np.arange(n) if kind == "count" else np.cumsum(rng.choice([0, 1, 1, 3], size=n))
        w = {"kind": kind, "size": 64, "slide": 8, "origin": 0}
        sp = tspec(w, aggs=[("avg", "x"), ("sum", "x"), ("count", None)],
                   group_by=[("k", 1, 5), ("v", d, 40), ("o", 1, 2)])
        data = stream(v=v, tau=tau, x=x, k=k, n=n)
        check(saber, oracle_lib, sp, data, task_bytes=32 * int(rng.choice([777, 5000, 20000])))


@pytest.mark.parametrize("case", ["minmax_having", "avg_two_keys_time", "g2048_tumbling"])
def test_win_wide(saber, oracle_lib, case):
    """k_win_wide (256 < C <= 2048 dense keys): one window per ticket, rows in key
    order, look-back per window; HAVING, min/max, ragged tasks."""
    if case == "minmax_having":
        spec, _ = workloads.c3(groups=700)
        spec["window"] = workloads.count_window(640, 64)
        spec["aggs"] = [("min", "a1"), ("max", "a3"), ("count", None)]
        spec["having"] = [(2, ">=", 2)]
        data = gen.generate("syn", 150000, 31, groups=700)
        tb = 32 * 9973
    elif case == "avg_two_keys_time":
        spec, g = workloads.c5b()
        spec["window"]["size"] = 20
        spec["window"]["slide"] = 2
        data = gen.generate("lrb", 1 << 18, 32, rate=512)
        tb = 32 * 30011
    else:
        spec, _ = workloads.c3(groups=2048)
        spec["window"] = workloads.count_window(512, 512)
        spec["aggs"] = [("avg", "a1"), ("sum", "a4")]
        data = gen.generate("syn", 1 << 17, 33, groups=2048)
        tb = 1 << 20
    check(saber, oracle_lib, spec, data, task_bytes=tb, result_slots=3)


# ------------------------------------------------- registered host memory ---
@pytest.mark.parametrize("mode", ["registered", "mixed"])
def test_register_host_direct_dma(saber, oracle_lib, mode):
    """The bench's end-to-end path: saber_register_host, then submits of whole
    tasks straight from the registered range (no copyin stage) plus a ragged tail,
    HOST result mode.  'mixed' interleaves unregistered (pageable, copyin) chunks
    and chunks that start mid-task."""
    import torch
    spec, g = workloads.c3(groups=64)
    spec["window"] = workloads.count_window(4096, 1024)
    n = (1 << 18) + 777
    data = gen.generate("syn", n, g["seed"], groups=64)
    exp = oracle_lib.run(spec, data, nthreads=8)
    pinned = torch.empty(len(data), dtype=torch.uint8).pin_memory() if mode == "mixed" else None
    host = np.frombuffer(data, np.uint8).copy()
    tb = 32 * 10000
    q = saber.Query(spec, task_bytes=tb, result_mode=saber.RESULTS_HOST, result_slots=4)
    if mode == "registered":
        q.register_host(host)            # cudaHostRegister of the caller's pages
        src = host
    else:
        pinned.numpy()[:] = host         # already page-locked (torch pinned memory)
        src = pinned.numpy()
        q.register_host(src)
    slices = []
    if mode == "registered":
        cuts = [0, 3 * tb, 5 * tb, len(data)]
    else:
        cuts = [0, tb + 32 * 5, 2 * tb + 32 * 5, 4 * tb, 4 * tb + 32 * 3, len(data)]
    unreg = np.frombuffer(data, np.uint8).copy()
    for c, (a, b) in enumerate(zip(cuts[:-1], cuts[1:])):
        chunk = src[a:b] if (mode == "registered" or c % 2 == 0) else unreg[a:b]
        off = 0
        while off < chunk.size:
            part = chunk[off:off + 3 * tb]
            st = q.submit(part)
            if st == saber.EAGAIN:
                slices.append(q.poll())
                continue
            assert st == 0, q.last_error()
            off += part.size
    while (st := q.finish()) == saber.EAGAIN:
        slices.append(q.poll())
    assert st == 0
    while (s := q.poll()) is not None:
        slices.append(s)
    q.close()
    compare(spec, saber.merge_slices(slices, q.m), exp)


def test_release_out_of_order_no_partial_submit(saber, oracle_lib):
    """Slices may be released in any order: a submit whose ring slots are not all
    free returns EAGAIN *without consuming* input, so retrying after the
    release continues the stream exactly (no tuple submitted twice or lost)."""
    spec, g = workloads.c3(groups=64)
    spec["window"] = workloads.count_window(2048, 512)
    tb = 32 * 4096
    n = 4096 * 9
    data = np.frombuffer(gen.generate("syn", n, g["seed"], groups=64), np.uint8)
    exp = oracle_lib.run(spec, data.tobytes(), nthreads=8)
    q = saber.Query(spec, task_bytes=tb, result_slots=4)
    for t in range(3):
        assert q.submit(data[t * tb:(t + 1) * tb]) == 0
    st0, r0 = q.poll_raw(-1)
    st1, r1 = q.poll_raw(-1)
    assert st0 == 0 and st1 == 0
    skip = set(range(int(r1.first_window), int(r1.first_window + r1.nwindows)))
    q.release(r1)                        # slot 1 free, slot 0 still held
    # the next two tasks need ring slots 3 and 0: slot 0 is held -> EAGAIN, nothing consumed
    assert q.submit(data[3 * tb:5 * tb]) == saber.EAGAIN
    q.release(r0)                        # slice 0 and 1 are not read: their windows are skipped
    skip |= set(range(int(r0.first_window), int(r0.first_window + r0.nwindows)))
    slices, off = [], 3 * tb
    while off < data.size:
        st = q.submit(data[off:off + 2 * tb])
        if st == saber.EAGAIN:
            slices.append(q.poll())
            continue
        assert st == 0, q.last_error()
        off += 2 * tb
    while (st := q.finish()) == saber.EAGAIN:
        slices.append(q.poll())
    assert st == 0
    while (sl := q.poll()) is not None:
        slices.append(sl)
    q.close()
    got = saber.merge_slices(slices, q.m)
    keep = ~np.isin(exp["win_id"], sorted(skip))
    rowkeep = np.repeat(keep, exp["win_nrows"])
    sub = {"win_id": exp["win_id"][keep], "win_ts": exp["win_ts"][keep], "win_nrows": exp["win_nrows"][keep],
           "keys": exp["keys"][rowkeep], "vals": [v[rowkeep] for v in exp["vals"]], "tuples": b""}
    assert len(sub["win_id"]) > 0
    compare(spec, got, sub)


# ------------------------------------------------------------ time gaps ---
def _cm_with_jump(n, seed, rate, at, jump, groups=4):
    d = gen.generate("cm", n, seed, rate=rate, groups=groups)
    ts = gen.column(d, "cm", "ts").copy()
    ts[at:] += jump
    return gen.with_column(d, "cm", "ts", ts)


@pytest.mark.parametrize("case", ["jump1e5_small_ring", "jump1e7_tumbling60", "jump1e6_w3600_s60", "jump_at_task_start"])
def test_time_gap_wider_than_ring(saber, oracle_lib, case):
    """A valid stream may jump in time by more than the pane ring holds (PAPER.md
    L345-352: any discrete, non-decreasing τ).  The task runs in rounds: data before
    the gap, the gap's windows as headers with nrows = 0 (reading A6) without
    touching the ring, then the data after it -- with the gap inside a task, at a
    task start, and a watermark far past the data."""
    spec, g = workloads.c4(rate=64)
    n = 60000
    kw = {}
    if case == "jump1e5_small_ring":
        data = _cm_with_jump(n, 51, 64, 31111, 100000)
        kw = dict(max_panes=2000)                      # ring of 4096 panes << the 10^5 s gap
        tbs = [64 * 7777, 64 * 30000, 64 * 100000]
    elif case == "jump1e7_tumbling60":
        spec["window"] = workloads.time_window(60, 60)
        data = _cm_with_jump(n, 52, 64, 20000, 10 ** 7)
        tbs = [64 * 9999, 64 * 100000]
    elif case == "jump1e6_w3600_s60":
        spec["window"] = workloads.time_window(3600, 60)
        data = _cm_with_jump(n, 53, 16, 40001, 10 ** 6)
        kw = dict(max_panes=600)
        tbs = [64 * 12345, 64 * 100000]
    else:
        data = _cm_with_jump(n, 54, 64, 30000, 50000)
        kw = dict(max_panes=1000)
        tbs = [64 * 30000, 64 * 15000]                 # the jump falls exactly on a task start
    ts = gen.column(data, "cm", "ts")
    for wm in (None, int(ts[-1]) + 5000):
        exp = oracle_lib.run(spec, data, watermark=wm, nthreads=8)
        for tb in tbs:
            got = run_product(saber, spec, data, task_bytes=tb, watermark=wm, result_slots=3, **kw)
            compare(spec, got, exp)
    assert (exp["win_nrows"] == 0).sum() > 1000          # the gap's empty windows are there


@pytest.mark.parametrize("npred", [16, 64])
def test_select_n_predicates(saber, oracle_lib, npred):
    """SELECT_n (Fig. 10a): n-1 extra always-true terms, same selectivity."""
    spec, g = workloads.c2(sel=0.3, npred=npred)
    data = gen.generate("syn", 1 << 18, g["seed"], rate=1)
    check(saber, oracle_lib, spec, data, task_bytes=(1 << 20) + 32 * 13)


# k_wb_rows + k_win_block_reg (FAST plans, one-pane slides, 32..256 dense keys):
# every template instance the planner can pick (C, K = (256/C)·{4, 8, 16}; key slices of 64
# for C = 256, K = 32 and C = 128, K = 64), two
# float sum fields (CM), a time window, ragged tasks whose windows span tasks
@pytest.mark.parametrize("case", ["c32_k32", "c64_k16", "c64_k64", "c128_k16", "c256_k8", "c256_k32", "c128_k64",
                                  "cm_nf2", "time_c64_k32"])
def test_win_block_reg(saber, oracle_lib, case):
    if case == "cm_nf2":
        spec, _ = workloads.c4(rate=64)
        spec["window"] = workloads.count_window(32 * 48, 48)
        spec["aggs"] = [("avg", "cpu"), ("sum", "ram"), ("count", None)]
        spec["group_by"] = [("category", 1, 64)]
        data = gen.generate("cm", 200000, 41, rate=64, groups=64)
        tb = 64 * 7919
    elif case == "time_c64_k32":
        spec, _ = workloads.c3(groups=64)
        spec["window"] = workloads.time_window(32, 1)
        data = gen.generate("syn", 300000, 42, rate=100, groups=64)
        tb = 32 * 12347
    else:
        c, k = (int(x[1:]) for x in case.split("_"))
        l = {32: 16, 64: 8, 128: 12, 256: 40}[c] if k != 64 else 8
        spec, _ = workloads.c3(groups=c)
        spec["window"] = workloads.count_window(k * l, l)
        spec["aggs"] = [("avg", "a1"), ("count", None), ("sum", "a1")]
        data = gen.generate("syn", 250000, 40 + c + k, groups=c)
        tb = 32 * 9973
    got, exp = check(saber, oracle_lib, spec, data, task_bytes=tb)
    assert len(exp["win_id"]) > 100
