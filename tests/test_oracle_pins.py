"""Pins for the CPU oracle (run with -m "not gpu").

Each test pins the oracle to something other than itself: values printed or
implied by the paper's worked examples (tests/golden/*.json, each with its
citation), closed forms, textbook routines (numpy reshape / convolve /
bincount), exact rational arithmetic, and an independent pure-Python brute
force (oracle/brute.py).  A plausible slip in oracle.cpp -- an off-by-one
window edge, a dropped tuple, a swapped operand, a wrong stream function --
fails at least one of them.
"""
from fractions import Fraction

import numpy as np
import pytest

from saber_inputs import gen, workloads
from tiny import TINY, golden, spec, stream


def sums(res, a=0):
    """Per-window value of aggregate a for a global (no GROUP BY) query; None if empty."""
    out = []
    for w in range(len(res["win_id"])):
        n = res["win_nrows"][w]
        out.append(None if n == 0 else res["vals"][a][res["win_rowoff"][w]])
    return out


# ---------------------------------------------------------------- goldens ----
@pytest.mark.parametrize("gid", ["G1", "G2"])
def test_fig2_membership(oracle_lib, gid):
    """Fig. 2 prose (L508-517): window membership via SUM of m = 2^i (a bitmask)."""
    g = golden(gid)
    sp = spec(g["window"], aggs=[("sum", "m"), ("sum", "v")])
    res = oracle_lib.run(sp, stream(v=g["tuples_v"]))
    masks = sums(res, 0)
    members = [[i for i in range(10) if (mk >> i) & 1] for mk in masks]
    assert members == g["expect_members"]
    assert sums(res, 1) == g["expect_sum"]
    # batch classification of Fig. 2 follows from membership: with 5-tuple batches a
    # window is complete in b1 iff all members < 5.
    tt = g["task_tuples"]
    cls0 = g["expect_task_classes"][0]
    complete = [j for j, m in enumerate(members) if max(m) < tt]
    assert complete == cls0["complete"]


def test_g3_tumbling(oracle_lib):
    g = golden("G3")
    res = oracle_lib.run(spec(g["window"], aggs=[("sum", "v")]), stream(v=g["tuples_v"]))
    assert sums(res) == g["expect_sum"]
    assert sum(g["expect_sum"]) == sum(range(1, 9))          # I1 on the golden itself


def test_g4_time_windows(oracle_lib):
    g = golden("G4")
    sp = spec(g["window"], aggs=[("count", None), ("sum", "v")])
    res = oracle_lib.run(sp, stream(v=g["tuples_v"], tau=g["tau"]))
    assert list(res["win_id"]) == list(range(6))
    assert sums(res, 0) == g["expect_count"]
    assert sums(res, 1) == g["expect_sum"]
    assert list(res["win_ts"]) == list(range(6))              # reading A7: ts = T0 + j*l


def test_g5_time_tumbling_empty_windows(oracle_lib):
    g = golden("G5")
    d = stream(v=g["tuples_v"], tau=g["tau"])
    r11 = oracle_lib.run(spec({"kind": "time", "size": 1, "slide": 1}, aggs=[("sum", "v")]), d)
    assert sums(r11) == g["w11_sum"]
    assert list(r11["win_nrows"]) == [0 if s is None else 1 for s in g["w11_sum"]]
    r22 = oracle_lib.run(spec({"kind": "time", "size": 2, "slide": 2}, aggs=[("sum", "v")]), d)
    assert sums(r22) == g["w22_sum"]


def _rows(res, nagg):
    out = []
    for w in range(len(res["win_id"])):
        o, n = res["win_rowoff"][w], res["win_nrows"][w]
        out.append({str(int(res["keys"][o + r][0])): [res["vals"][a][o + r] for a in range(nagg)]
                    for r in range(n)})
    return out


def test_g6_groupby_exact(oracle_lib):
    g = golden("G6")
    sp = spec(g["window"], aggs=[("sum", "x"), ("count", None), ("avg", "x")], group_by=[("k", 1, 0)])
    res = oracle_lib.run(sp, stream(x=g["x"], k=g["key"]))
    got = _rows(res, 3)
    assert got == [{k: [float(v[0]), int(v[1]), float(v[2])] for k, v in w.items()} for w in g["expect"]]
    # rows are ascending by key inside each window (reading A8)
    for w in range(len(res["win_id"])):
        o, n = res["win_rowoff"][w], res["win_nrows"][w]
        assert list(res["keys"][o:o + n, 0]) == sorted(res["keys"][o:o + n, 0])


def test_g7_istream(oracle_lib):
    g = golden("G7")
    sp = spec(g["window"], where=[("o", "==", 1)], project=["v"])
    res = oracle_lib.run(sp, stream(v=g["tuples_v"]))
    assert list(np.frombuffer(res["tuples"], dtype=np.int32)) == g["expect_v"]


def test_g9_having(oracle_lib):
    g6, g9 = golden("G6"), golden("G9")
    sp = spec(g6["window"], aggs=[("avg", "x")], group_by=[("k", 1, 0)], having=[(0, "<", 1.0)])
    res = oracle_lib.run(sp, stream(x=g6["x"], k=g6["key"]))
    assert _rows(res, 1) == [{k: [v] for k, v in w.items()} for w in g9["expect"]]
    assert list(res["win_id"]) == [0, 1, 2, 3]               # headers kept for empty results (A6)


def test_g8_panes_reduce_to_g4(oracle_lib):
    """G8: an w(s,l) aggregate equals the fold of its g-long panes (I9 on the golden)."""
    g4, g8 = golden("G4"), golden("G8")
    d = stream(v=g4["tuples_v"], tau=g4["tau"])
    panes = oracle_lib.run(spec({"kind": "time", "size": 1, "slide": 1}, aggs=[("count", None)]), d)
    cnt = [0 if c is None else c for c in sums(panes)]
    assert list(np.concatenate([[0], np.cumsum(cnt)])) == g8["pane_off"]


# --------------------------------------------------------- closed forms ------
@pytest.mark.parametrize("n,s,l", [(0, 4, 2), (3, 4, 2), (4, 4, 2), (100, 7, 3), (1000, 32, 32), (999, 40, 1)])
def test_count_window_closed_form(oracle_lib, n, s, l):
    """I2: W = floor((N-s)/l)+1 for N >= s (from m = k+s-1, next start k+l, L370-372)."""
    d = stream(v=np.arange(n), n=n)
    w = oracle_lib.num_windows(spec({"kind": "count", "size": s, "slide": l}, aggs=[("count", None)]), d)
    assert w == (0 if n < s else (n - s) // l + 1)


@pytest.mark.parametrize("rate,s,l", [(1, 5, 1), (3, 10, 2), (7, 7, 7), (4, 9, 3)])
def test_time_window_closed_form(oracle_lib, rate, s, l):
    """I2 for constant rate R (tau_i = floor(i/R)): W = floor((floor((N-1)/R)+1-s)/l)+1."""
    n = 200
    tau = np.arange(n) // rate
    d = stream(tau=tau, n=n)
    res = oracle_lib.run(spec({"kind": "time", "size": s, "slide": l}, aggs=[("count", None)]), d)
    expect = ((n - 1) // rate + 1 - s) // l + 1
    assert len(res["win_id"]) == expect
    # every window of a constant-rate stream holds exactly s*R tuples (count = s*R)
    assert all(c == s * rate for c in sums(res))


# ------------------------------------------------------------- invariants ----
def _syn(n, seed=11, groups=8, rate=1):
    return gen.generate("syn", n, seed=seed, rate=rate, groups=groups)


def _syn_spec(window, **kw):
    sp, _ = workloads.c1()
    sp["window"] = dict(window)
    sp["aggs"] = kw.get("aggs", [])
    sp["group_by"] = kw.get("group_by", [])
    sp["where"] = kw.get("where", [])
    sp["project"] = kw.get("project", [])
    sp["having"] = kw.get("having", [])
    return sp


def test_tumbling_matches_numpy_reshape(oracle_lib):
    """Tumbling SUM/MIN/MAX/COUNT/AVG == numpy reshape reductions (textbook routine)."""
    n, s = 5000, 64
    d = _syn(n)
    a1 = gen.column(d, "syn", "a1").astype(np.float64)
    a3 = gen.column(d, "syn", "a3").astype(np.int64)
    sp = _syn_spec({"kind": "count", "size": s, "slide": s},
                   aggs=[("sum", "a3"), ("min", "a1"), ("max", "a1"), ("count", None), ("sum", "a1"),
                         ("avg", "a3")])
    res = oracle_lib.run(sp, d)
    W = n // s
    assert len(res["win_id"]) == W
    x3 = a3[:W * s].reshape(W, s)
    x1 = a1[:W * s].reshape(W, s)
    assert np.array_equal(res["vals"][0], x3.sum(1))
    assert np.array_equal(res["vals"][1], x1.min(1))
    assert np.array_equal(res["vals"][2], x1.max(1))
    assert np.array_equal(res["vals"][3], np.full(W, s))
    np.testing.assert_allclose(res["vals"][4], x1.sum(1), rtol=1e-12)
    np.testing.assert_allclose(res["vals"][5], x3.sum(1) / s, rtol=1e-15)


def test_sliding_sum_matches_convolve(oracle_lib):
    """Sliding integer SUM == numpy.convolve(x, ones(s))[s-1::l] (exact)."""
    n, s, l = 3000, 48, 5
    d = _syn(n)
    a3 = gen.column(d, "syn", "a3").astype(np.int64)
    res = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l}, aggs=[("sum", "a3")]), d)
    ref = np.convolve(a3, np.ones(s, dtype=np.int64))[s - 1:n:l]
    assert np.array_equal(res["vals"][0], ref)


def test_groupby_matches_bincount(oracle_lib):
    """GROUP BY COUNT/SUM per window == numpy.bincount(key, weights) on the window slice."""
    n, s, l, G = 4000, 256, 128, 16
    d = _syn(n, groups=G)
    key = gen.column(d, "syn", "a2")
    a3 = gen.column(d, "syn", "a3").astype(np.int64)
    sp = _syn_spec({"kind": "count", "size": s, "slide": l}, aggs=[("count", None), ("sum", "a3")],
                   group_by=[("a2", 1, 0)])
    res = oracle_lib.run(sp, d)
    for j in range(len(res["win_id"])):
        sl = slice(j * l, j * l + s)
        cnt = np.bincount(key[sl], minlength=G)
        sm = np.zeros(G, dtype=np.int64)
        np.add.at(sm, key[sl], a3[sl])
        present = np.nonzero(cnt)[0]
        o, nr = res["win_rowoff"][j], res["win_nrows"][j]
        assert np.array_equal(res["keys"][o:o + nr, 0], present)
        assert np.array_equal(res["vals"][0][o:o + nr], cnt[present])
        assert np.array_equal(res["vals"][1][o:o + nr], sm[present])


def test_invariants_random(oracle_lib):
    """I1 tumbling totals, I3 sum of group counts = s, I5 G=1 == global,
    I6 AVG*COUNT ~ SUM and MIN <= AVG <= MAX, I9 pane composition."""
    rng = np.random.default_rng(5)
    for trial in range(6):
        n = int(rng.integers(2000, 6000))
        G = int(rng.choice([1, 3, 16]))
        d = _syn(n, seed=100 + trial, groups=G)
        a3 = gen.column(d, "syn", "a3").astype(np.int64)
        g = int(rng.choice([8, 16, 32]))
        K = int(rng.integers(1, 5))
        s, l = g * K, g * int(rng.integers(1, K + 1))
        # I1
        rt = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": s}, aggs=[("sum", "a3")]), d)
        W = n // s
        assert int(np.sum(rt["vals"][0])) == int(a3[:W * s].sum())
        # I3 + I6
        sp = _syn_spec({"kind": "count", "size": s, "slide": l},
                       aggs=[("count", None), ("sum", "a1"), ("avg", "a1"), ("min", "a1"), ("max", "a1")],
                       group_by=[("a2", 1, 0)])
        r = oracle_lib.run(sp, d)
        for j in range(len(r["win_id"])):
            o, nr = r["win_rowoff"][j], r["win_nrows"][j]
            assert int(r["vals"][0][o:o + nr].sum()) == s
        np.testing.assert_allclose(r["vals"][2] * r["vals"][0], r["vals"][1], rtol=1e-12)
        assert np.all(r["vals"][3] <= r["vals"][2] + 1e-12) and np.all(r["vals"][2] <= r["vals"][4] + 1e-12)
        # I5: grouping by a constant column (G=1 stream) == no GROUP BY
        if G == 1:
            rg = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l}, aggs=[("sum", "a3")],
                                          group_by=[("a2", 1, 0)]), d)
            r0 = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l}, aggs=[("sum", "a3")]), d)
            assert np.array_equal(rg["vals"][0], r0["vals"][0])
        # I9: w(s,l) SUM == sum of its K tumbling w(g,g) pane sums
        rs = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l}, aggs=[("sum", "a3")]), d)
        rp = oracle_lib.run(_syn_spec({"kind": "count", "size": g, "slide": g}, aggs=[("sum", "a3")]), d)
        P = rp["vals"][0]
        L = l // g
        for j in range(len(rs["win_id"])):
            assert rs["vals"][0][j] == P[j * L:j * L + K].sum()


def test_time_on_positions_equals_count(oracle_lib):
    """I4: time windows over tau_i = i are exactly count windows (bit-exact, floats too)."""
    n = 3000
    d = _syn(n, groups=8)
    for s, l in [(100, 10), (64, 64), (1, 1), (37, 5)]:
        aggs = [("sum", "a1"), ("avg", "a1"), ("min", "a3"), ("max", "a1"), ("count", None)]
        rc = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l}, aggs=aggs,
                                      group_by=[("a2", 1, 0)]), d)
        rt = oracle_lib.run(_syn_spec({"kind": "time", "size": s, "slide": l}, aggs=aggs,
                                      group_by=[("a2", 1, 0)]), d, watermark=n)
        for key in ("win_id", "win_ts", "win_nrows", "keys"):
            assert np.array_equal(rc[key], rt[key])
        for a in range(len(aggs)):
            assert np.array_equal(rc["vals"][a].view(np.uint64), rt["vals"][a].view(np.uint64))


def test_istream_identity_and_counts(oracle_lib):
    """I7 (sigma true, pi = all columns => output = covered input bytes) and
    I11 (#IStream rows = #covered selected tuples); also w(1,1) per-tuple (I8)."""
    n = 2000
    d = _syn(n)
    allcols = [c for c, _, _ in gen.SCHEMAS["syn"]["cols"]]
    for s, l in [(64, 8), (100, 100), (1, 1), (50, 49)]:
        r = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l}, project=allcols), d)
        W = (n - s) // l + 1
        covered = (W - 1) * l + s
        assert r["tuples"] == d[:covered * 32]
        a3 = gen.column(d, "syn", "a3")
        th = 1 << 30
        rs = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l},
                                      where=[("a3", "<", th)], project=["a3"]), d)
        got = np.frombuffer(rs["tuples"], dtype=np.int32)
        exp = a3[:covered][a3[:covered] < th]
        assert np.array_equal(got, exp)


def test_float_sum_accuracy_exact_rationals(oracle_lib):
    """fp64 SUM in the oracle is within 1e-12 of the exact rational sum (Fraction)."""
    n, s, l = 6000, 4000, 500
    d = _syn(n)
    a1 = gen.column(d, "syn", "a1")
    r = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l}, aggs=[("sum", "a1")]), d)
    for j in range(len(r["win_id"])):
        exact = sum((Fraction(float(x)) for x in a1[j * l:j * l + s]), Fraction(0))
        assert abs(Fraction(float(r["vals"][0][j])) - exact) <= Fraction(1, 10 ** 12) * exact


def test_threads_do_not_change_results(oracle_lib):
    """Parallelism is across windows only: 1 and 4 threads give identical bytes."""
    n = 20000
    d = _syn(n, groups=64)
    sp = _syn_spec({"kind": "count", "size": 512, "slide": 64}, aggs=[("avg", "a1"), ("max", "a3")],
                   group_by=[("a2", 1, 0)])
    r1 = oracle_lib.run(sp, d, nthreads=1)
    r4 = oracle_lib.run(sp, d, nthreads=4)
    for key in ("win_id", "win_nrows", "keys"):
        assert np.array_equal(r1[key], r4[key])
    for a in range(2):
        assert np.array_equal(r1["vals"][a].view(np.uint64), r4["vals"][a].view(np.uint64))


def test_window_sampling_matches_full(oracle_lib):
    """The sampled-window entry point returns exactly the full run's windows."""
    n = 5000
    d = _syn(n, groups=16, rate=7)
    sp = _syn_spec({"kind": "time", "size": 50, "slide": 3}, aggs=[("sum", "a1"), ("count", None)],
                   group_by=[("a2", 1, 0)])
    full = oracle_lib.run(sp, d)
    ids = [0, 5, 17, len(full["win_id"]) - 1]
    part = oracle_lib.run(sp, d, windows=ids)
    for k, j in enumerate(ids):
        o, nr = full["win_rowoff"][j], full["win_nrows"][j]
        po, pn = part["win_rowoff"][k], part["win_nrows"][k]
        assert nr == pn
        assert np.array_equal(full["keys"][o:o + nr], part["keys"][po:po + pn])
        assert np.array_equal(full["vals"][0][o:o + nr], part["vals"][0][po:po + pn])


def test_errors(oracle_lib):
    """Non-monotone timestamps (L347-349) and negative timestamps (A24) are rejected."""
    with pytest.raises(oracle_lib.OracleError) as e:
        oracle_lib.run(spec({"kind": "time", "size": 2, "slide": 1}, aggs=[("count", None)]),
                       stream(tau=[0, 2, 1]))
    assert e.value.code == -1
    with pytest.raises(oracle_lib.OracleError) as e:
        oracle_lib.run(spec({"kind": "time", "size": 2, "slide": 1}, aggs=[("count", None)]),
                       stream(tau=[-1, 2]))
    assert e.value.code == -22
    # empty input and N < s: no windows, no output
    r = oracle_lib.run(spec({"kind": "count", "size": 4, "slide": 1}, aggs=[("count", None)]), b"")
    assert len(r["win_id"]) == 0
    r = oracle_lib.run(spec({"kind": "count", "size": 4, "slide": 1}, aggs=[("count", None)]),
                       stream(v=[1, 2, 3]))
    assert len(r["win_id"]) == 0


def test_int64_sum_overflow_detected(oracle_lib):
    """SUM over an I64 column is checked (reading A14): a window whose exact sum
    leaves [-2^63, 2^63) makes the oracle report OQ_EOVERFLOW (-75); sums that end
    exactly on the representable boundary do not."""
    def run(m):
        a = np.zeros(len(m), dtype=[("ts", "<i8"), ("v", "<i4"), ("x", "<f4"), ("m", "<i8"),
                                    ("k", "<i4"), ("o", "<i4")])
        a["ts"] = np.arange(len(m))
        a["m"] = m
        return oracle_lib.run(spec({"kind": "count", "size": 2, "slide": 2}, aggs=[("sum", "m")]), a.tobytes())
    big = 1 << 62
    r = run([big, big - 1, -big, -big])                  # 2^63 - 1 and -2^63: both exact
    assert list(r["vals"][0]) == [(1 << 63) - 1, -(1 << 63)]
    for m in ([big, big], [-big, -big - 1], [1, 2, big, big]):
        with pytest.raises(oracle_lib.OracleError) as e:
            run(m)
        assert e.value.code == -75, m


def test_istream_rows_per_window(oracle_lib):
    """IStream headers (reading A9): window j's row count is the number of selected
    tuples in the position segment W_j \\ W_{j-1} = [(j-1)·l + s, j·l + s) (j >= 1;
    W_0 whole), counted here with numpy; header ts = τ of position j·l (A7)."""
    n = 3000
    d = _syn(n)
    a3 = gen.column(d, "syn", "a3")
    ts = gen.column(d, "syn", "ts")
    th = 1 << 30
    for s, l in [(64, 8), (100, 100), (1, 1), (50, 49), (7, 3)]:
        r = oracle_lib.run(_syn_spec({"kind": "count", "size": s, "slide": l},
                                     where=[("a3", "<", th)], project=["a3"]), d)
        W = (n - s) // l + 1
        sel = (a3 < th).astype(np.int64)
        exp = [int(sel[0:s].sum())] + [int(sel[(j - 1) * l + s:j * l + s].sum()) for j in range(1, W)]
        assert list(r["win_nrows"]) == exp
        assert list(r["win_ts"]) == [int(ts[j * l]) for j in range(W)]


# ------------------------------------------------------------------ θ-join ---
def _jspec(w, theta, p1=("ts", "a1"), p2=("a1", "a2")):
    sch = gen.SCHEMAS["syn"]
    return {"schema1": sch, "schema2": sch, "window": w, "theta": list(theta),
            "project1": list(p1), "project2": list(p2)}


def test_join_matches_brute_force(oracle_lib):
    """The oracle's windowed θ-join equals an independent Python formulation
    (oracle/brute.py: 1-based windows, sets of matching pairs) byte for byte."""
    from oracle.brute import brute_join
    rng = np.random.default_rng(5)
    for _ in range(40):
        n1, n2 = int(rng.integers(0, 40)), int(rng.integers(0, 40))
        s = int(rng.integers(1, 9))
        l = int(rng.integers(1, s + 1))
        d1 = bytearray(gen.generate("syn", n1, int(rng.integers(1, 99)), groups=3))
        d2 = bytearray(gen.generate("syn", n2, int(rng.integers(1, 99)), groups=3))
        ops = ["<", "<=", ">", ">=", "==", "!="]
        theta = [(str(rng.choice(["a2", "a3", "a1"])), str(rng.choice(ops)), str(rng.choice(["a2", "a4", "a1"])))
                 for _ in range(int(rng.integers(0, 3)))]
        js = _jspec({"kind": "count", "size": s, "slide": l}, theta)
        got = oracle_lib.join_run(js, bytes(d1), bytes(d2))
        exp = brute_join(js, bytes(d1), bytes(d2))
        assert list(got["win_id"]) == [j for j, _, _ in exp]
        assert list(got["win_ts"]) == [ts for _, ts, _ in exp]
        assert list(got["win_nrows"]) == [len(r) for _, _, r in exp]
        assert got["tuples"] == b"".join(b"".join(r) for _, _, r in exp)


def test_join_cross_product_and_equijoin_counts(oracle_lib):
    """Closed forms: with no θ term every window emits s^2 pairs (the window cross
    product); an equi-join on a key emits sum_k c1(k)·c2(k) pairs per window
    (numpy bincount of each side's window)."""
    n, s, l = 3000, 64, 48
    d1 = gen.generate("syn", n, 21, groups=7)
    d2 = gen.generate("syn", n, 22, groups=7)
    r = oracle_lib.join_run(_jspec({"kind": "count", "size": s, "slide": l}, []), d1, d2)
    W = (n - s) // l + 1
    assert list(r["win_nrows"]) == [s * s] * W
    r = oracle_lib.join_run(_jspec({"kind": "count", "size": s, "slide": l}, [("a2", "==", "a2")]), d1, d2)
    k1, k2 = gen.column(d1, "syn", "a2"), gen.column(d2, "syn", "a2")
    exp = [int((np.bincount(k1[j * l:j * l + s], minlength=7) * np.bincount(k2[j * l:j * l + s], minlength=7)).sum())
           for j in range(W)]
    assert list(r["win_nrows"]) == exp
