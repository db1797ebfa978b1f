"""Float robustness of every window-assembly plan.

The benchmark generators emit u24 values (multiples of 2^-24 in [0,1)), whose
fp64 sums are exact -- they cannot expose cancellation in plans that slide a
window state by adding entering and subtracting expiring partials.  Here the
aggregated column is non-negative, non-dyadic and log-uniform over 18 decades
(1e-6 .. 1e12, saber_inputs.gen.wide_f32), so a key whose window once held a
1e12 value and now holds only tiny ones exposes any error proportional to the
state's history.  Every plan must stay within the north_star tolerance
(|g - o| <= 1e-5 |o|, fp64 on both sides, PAPER.md-independent reading A12).
"""
import numpy as np
import pytest

from parity import compare
from saber_inputs import gen, workloads

pytestmark = pytest.mark.gpu

WINDOW_KINDS = {1: "vh", 2: "win_block", 3: "bucket", 4: "hash", 5: "slab", 6: "win_wide"}


@pytest.fixture(scope="module")
def saber():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_sigmod_koliousiswfwcp16_b200 import saber as S
    return S


def _syn_wide(n, seed, groups, lo=-6.0, hi=12.0):
    d = gen.generate("syn", n, seed, groups=groups)
    return gen.with_column(d, "syn", "a1", gen.wide_f32(seed, 0, n, lo, hi))


def _case(name):
    if name == "bucket_g20000":
        spec, _ = workloads.c3(groups=20000)
        spec["window"] = workloads.count_window(4096, 512)
        spec["aggs"] = [("avg", "a1"), ("sum", "a1"), ("count", None)]
        return spec, _syn_wide(150000, 41, 20000), 1 << 20, "bucket"
    if name == "bucket_mid_g4096":
        spec, _ = workloads.c3(groups=4096)
        spec["window"] = workloads.count_window(8192, 1024)
        return spec, _syn_wide(200000, 42, 4096), 1 << 20, "bucket"
    if name == "hash_undeclared":
        spec, _ = workloads.c3(groups=3000, declare_domain=False)
        spec["window"] = workloads.count_window(2048, 256)
        spec["aggs"] = [("sum", "a1"), ("avg", "a1")]
        return spec, _syn_wide(120000, 43, 3000), 1 << 20, "hash"
    if name == "slab_time":
        spec, _ = workloads.c3(groups=20000)
        spec["window"] = workloads.time_window(3000, 500)
        spec["aggs"] = [("sum", "a1"), ("count", None)]
        return spec, _syn_wide(100000, 44, 20000), 1 << 20, "slab"
    if name == "dense_g64":
        spec, _ = workloads.c3(groups=64)
        spec["window"] = workloads.count_window(4096, 256)
        return spec, _syn_wide(150000, 45, 64), 1 << 20, None
    if name == "wide_g700":
        spec, _ = workloads.c3(groups=700)
        spec["window"] = workloads.count_window(8192, 512)
        return spec, _syn_wide(150000, 46, 700), 1 << 20, None
    if name == "global_sum":
        spec, _ = workloads.c1("sum")
        spec["window"] = workloads.count_window(5000, 100)
        return spec, _syn_wide(100000, 47, 64), 1 << 20, None
    raise KeyError(name)


@pytest.mark.parametrize("name", ["bucket_g20000", "bucket_mid_g4096", "hash_undeclared", "slab_time",
                                  "dense_g64", "wide_g700", "global_sum"])
def test_wide_range_floats(saber, oracle_lib, name):
    spec, data, tb, want = _case(name)
    exp = oracle_lib.run(spec, data, nthreads=8)
    q = saber.Query(spec, task_bytes=tb)
    got = q.run(data)
    kind = WINDOW_KINDS.get(q.stats()["window_kind"])
    q.close()
    if want:
        assert kind == want, f"plan is {kind}, expected {want}"
    compare(spec, got, exp)
    print(f"{name}: plan {kind}, {len(exp['win_id'])} windows, {int(exp['win_nrows'].sum())} rows compared")


def test_magnitude_swing_single_key(saber, oracle_lib):
    """Adversarial: one key holds 1e15 once and afterwards only values ~1 while its
    window count never returns to 0 (the sliding state's history dwarfs its value)."""
    for groups, w in ((20000, workloads.count_window(2048, 256)), (64, workloads.count_window(2048, 256))):
        spec, _ = workloads.c3(groups=groups)
        spec["window"] = w
        n = 60000
        d = gen.generate("syn", n, 48, groups=groups)
        keys = gen.column(d, "syn", "a2").copy()
        vals = (1.0 + gen.wide_f32(48, 0, n, -3, -1)).astype(np.float32)
        keys[::3] = 7                       # key 7 is dense in every window
        vals[1000] = 1e15
        keys[1000] = 7
        d = gen.with_column(gen.with_column(d, "syn", "a2", keys), "syn", "a1", vals)
        exp = oracle_lib.run(spec, d, nthreads=8)
        q = saber.Query(spec, task_bytes=1 << 20)
        got = q.run(d)
        q.close()
        compare(spec, got, exp)
