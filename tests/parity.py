"""Comparison of a product result with the oracle's.

* bit-exact: window ids, header timestamps, rows per window, keys, COUNT,
  integer SUM/MIN/MAX, float MIN/MAX, IStream bytes;
* float SUM / AVG: |gpu - oracle| <= 1e-5 * |oracle| (fp64 on both sides,
  the tolerance north_star states);
* rows inside a window have no specified order: both sides are sorted by key.
"""
import numpy as np

RTOL = 1e-5


def _float_agg(spec, a):
    fn, col = spec["aggs"][a]
    if fn == "avg":
        return True
    if fn == "count":
        return False
    ctype = {c[0]: c[1] for c in spec["schema"]["cols"]}[col]
    return ctype in ("f32", "f64")


def compare(spec, got, exp, rtol=RTOL):
    """Raise AssertionError with a precise message on the first mismatch."""
    assert np.array_equal(got["win_id"], exp["win_id"]), \
        f"window ids differ: got {got['win_id'][:8]}.. ({len(got['win_id'])}) exp {exp['win_id'][:8]}.. ({len(exp['win_id'])})"
    # headers: σ/π (IStream) windows too -- nrows counts the projected tuples of
    # W_j \ W_{j-1} (reading A9), ts is reading A7
    assert np.array_equal(got["win_ts"], exp["win_ts"]), \
        f"window timestamps differ at {np.nonzero(got['win_ts'] != exp['win_ts'])[0][:5]}"
    assert np.array_equal(got["win_nrows"], exp["win_nrows"]), \
        f"rows per window differ at {np.nonzero(got['win_nrows'] != exp['win_nrows'])[0][:5]}"
    if not spec.get("aggs"):
        assert got["tuples"] == exp["tuples"], \
            f"IStream bytes differ ({len(got['tuples'])} vs {len(exp['tuples'])} bytes)"
        return
    nk = len(spec.get("group_by", []))
    na = len(spec["aggs"])
    nrows = int(exp["win_nrows"].sum())
    gk = np.stack([k.astype(np.int64) for k in got["keys"]], 1) if nk else np.zeros((nrows, 0), np.int64)
    ek = exp["keys"]
    # sort rows by (window, key...) on both sides
    wid = np.repeat(np.arange(len(exp["win_nrows"])), exp["win_nrows"])
    def order(keys):
        cols = [keys[:, i] for i in reversed(range(nk))] + [wid]
        return np.lexsort(cols) if nrows else np.zeros(0, np.int64)
    og, oe = order(gk), order(ek)
    assert np.array_equal(gk[og], ek[oe]), "group keys differ"
    for a in range(na):
        g, e = got["vals"][a][og], exp["vals"][a][oe]
        fn = spec["aggs"][a][0]
        if _float_agg(spec, a) and fn in ("sum", "avg"):
            err = np.abs(g.astype(np.float64) - e)
            bad = err > rtol * np.abs(e)
            assert not bad.any(), f"agg {a} ({fn}) exceeds rtol {rtol}: worst rel " \
                f"{(err / np.maximum(np.abs(e), 1e-300)).max():.3e} at row {np.argmax(bad)}"
        else:
            assert np.array_equal(g.view(np.uint64), e.view(np.uint64)), f"agg {a} ({fn}) not bit-exact"
