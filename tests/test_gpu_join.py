"""GPU parity of the windowed θ-join (§5.4):
the CUDA path through the C ABI against the oracle's literal pair loops, byte
for byte (window ids, ts, pairs per window, and the pair rows in (a, b) order)."""
import numpy as np
import pytest

from saber_inputs import gen, workloads

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def saber():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    from paper_conf_sigmod_koliousiswfwcp16_b200 import saber as S
    return S


def _check(S, oracle_lib, js, d1, d2, batch, **kw):
    exp = oracle_lib.join_run(js, d1, d2, nthreads=8)
    j = S.Join(js, task_bytes=max(batch, 1) * js["schema1"]["tuple_bytes"], **kw)
    got = j.run(d1, d2, batch)
    j.close()
    assert np.array_equal(got["win_id"], exp["win_id"])
    assert np.array_equal(got["win_ts"], exp["win_ts"])
    assert np.array_equal(got["win_nrows"], exp["win_nrows"]), \
        f"pairs per window differ at {np.nonzero(got['win_nrows'] != exp['win_nrows'])[0][:5]}"
    assert got["tuples"] == exp["tuples"]
    return exp


@pytest.mark.parametrize("r", [1, 2, 4, 7])
def test_join_r_tumbling(saber, oracle_lib, r):
    """JOIN_r over two Syn streams, ω(1024, 1024) (the paper's ω32KB,32KB)."""
    js, g = workloads.join_r(r=r)
    n = 1 << 14
    d1 = gen.generate("syn", n, g["seed1"])
    d2 = gen.generate("syn", n, g["seed2"])
    exp = _check(saber, oracle_lib, js, d1, d2, 4096)
    assert exp["win_nrows"].sum() > 0


@pytest.mark.parametrize("case", ["sliding_ragged", "equi_key", "float_theta", "no_theta_small", "istream_like_slide1"])
def test_join_windows(saber, oracle_lib, case):
    """Sliding windows spanning tasks (carry of both streams), ragged batches,
    equi-joins on a key, float comparisons, the cross product, slide 1."""
    sch = gen.SCHEMAS["syn"]
    base = {"schema1": sch, "schema2": sch, "project1": ["ts", "a1"], "project2": ["a1", "a2"]}
    if case == "sliding_ragged":
        js = dict(base, window=workloads.count_window(700, 300), theta=[("a3", "<", "a4"), ("a5", ">", "a6")])
        n, batch = 9000, 1777
    elif case == "equi_key":
        js = dict(base, window=workloads.count_window(512, 128), theta=[("a2", "==", "a2")])
        n, batch = 6000, 1000
    elif case == "float_theta":
        js = dict(base, window=workloads.count_window(300, 300), theta=[("a1", "<", "a1"), ("a2", "!=", "a2")])
        n, batch = 5000, 333
    elif case == "no_theta_small":
        js = dict(base, window=workloads.count_window(40, 16), theta=[])
        n, batch = 2000, 97
    else:
        js = dict(base, window=workloads.count_window(64, 1), theta=[("a3", "<=", "a3")])
        n, batch = 3000, 1000
    d1 = gen.generate("syn", n, 31, groups=16)
    d2 = gen.generate("syn", n, 32, groups=16)
    _check(saber, oracle_lib, js, d1, d2, batch)


def test_join_device_submit_and_device_results(saber, oracle_lib):
    """Device batches (saber_join_submit_device) and DEVICE result mode."""
    import torch
    from cuda.bindings import runtime as rt
    js, g = workloads.join_r(r=3, size=1024, slide=512)
    n = 1 << 13
    d1 = gen.generate("syn", n, 41)
    d2 = gen.generate("syn", n, 42)
    exp = oracle_lib.join_run(js, d1, d2, nthreads=8)
    t1 = torch.from_numpy(np.frombuffer(d1, np.uint8).copy()).cuda()
    t2 = torch.from_numpy(np.frombuffer(d2, np.uint8).copy()).cuda()
    j = saber.Join(js, task_bytes=2048 * 32, result_mode=saber.RESULTS_DEVICE, result_slots=4)
    stream = torch.cuda.current_stream().cuda_stream
    for off in range(0, n, 2048):                     # 4 tasks, 4 result slots
        assert j.submit_device(t1.data_ptr() + off * 32, t2.data_ptr() + off * 32, 2048, stream) == 0, j.last_error()
    out, nrows = b"", 0
    while True:
        st, r = j.poll_raw(-1)
        if st != 0:
            break
        assert r.on_device
        if r.ntuples:
            host = np.empty(r.ntuples * r.tuple_bytes, np.uint8)
            (err,) = rt.cudaMemcpy(host.ctypes.data, int(r.tuples), host.size, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost)
            assert int(err) == 0
            out += host.tobytes()
        nrows += r.ntuples
        j.release(r)
    j.close()
    assert nrows == int(exp["win_nrows"].sum())
    assert out == exp["tuples"]
