"""Multi-GPU partitioning host logic on CPU (world_size 2 and 3, gloo).

Each rank owns a contiguous partition of one global stream, receives its halo
from the predecessor through torch.distributed P2P (parallel.exchange_halo), and
must emit exactly the windows [closed(r-1), closed(r)).  The per-rank window
evaluation is emulated with the oracle on [halo ++ partition] (the GPU does this
in production); the concatenation over ranks must equal the oracle over the
whole stream -- i.e. the plan + exchange lose and duplicate nothing.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from saber_inputs import gen, workloads


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _case(name):
    if name == "count":
        spec, g = workloads.c3(groups=16)
        spec["window"] = workloads.count_window(96, 32)
        return spec, dict(g, n=3000)
    if name == "count_tumbling":
        spec, g = workloads.c1("sum")
        spec["window"] = workloads.count_window(64, 64)
        return spec, dict(g, n=2000)
    spec, g = workloads.c4(rate=7)
    spec["window"] = workloads.time_window(20, 3)
    return spec, dict(g, n=3000)


def oracle_plan(spec, part, begin, n):
    """(windows closed by the partition's last tuple, first global position its
    successor needs), from the oracle: the closed-window count of the stream
    prefix and the first tuple of the next window (test-side twin of
    saber_partition_plan; the partition holds every tuple from begin)."""
    import oracle
    w = spec["window"]
    tb = spec["schema"]["tuple_bytes"]
    data = part.numpy()
    if w["kind"] == "count":
        closed = (begin + n - w["size"]) // w["slide"] + 1 if begin + n >= w["size"] else 0
        return closed, closed * w["slide"]
    ts = np.ascontiguousarray(data.reshape(-1, tb)[:, :8]).view(np.int64).reshape(-1)
    # windows closed by the last tuple: end <= τ_last (a tuple at or past the end arrived, reading A3)
    closed = int(oracle.num_windows(spec, data.tobytes(), watermark=int(ts[-1])))
    B = w.get("origin", 0) + closed * w["slide"]
    return closed, begin + int(np.searchsorted(ts, B, side="left"))


def _worker(rank, world, port, name, outq):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from paper_conf_sigmod_koliousiswfwcp16_b200.parallel import exchange_halo, partition_bounds
    spec, g = _case(name)
    N = g["n"]
    b, e = partition_bounds(N, world, rank)
    n = e - b
    data = gen.generate_array(g["kind"], n, g["seed"], i0=b, rate=g["rate"], groups=g["groups"]).reshape(-1)
    part = torch.from_numpy(data.copy())
    halo, first_window, base_index = exchange_halo(spec, part, b, n, rank, world, plan=oracle_plan)
    local = np.concatenate([halo.numpy(), data])
    tb = spec["schema"]["tuple_bytes"]
    # emulate the device pass on this rank with the oracle
    res = oracle.run(spec, local.tobytes())
    closed = oracle_plan(spec, part, b, n)[0] if rank < world - 1 else None
    w = spec["window"]
    ids = res["win_id"] + (base_index // w["slide"] if w["kind"] == "count" else 0)
    keep = ids >= first_window
    if closed is not None:
        keep &= ids < closed
    rows = []
    for k in np.nonzero(keep)[0]:
        o, nr = res["win_rowoff"][k], res["win_nrows"][k]
        rows.append((int(ids[k]), [tuple(res["keys"][r]) for r in range(o, o + nr)],
                     [tuple(v[r].item() for v in res["vals"]) for r in range(o, o + nr)]))
    assert len(local) == (len(data) + halo.numel()) and len(local) % tb == 0
    outq.put((rank, rows))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("name,world", [("count", 2), ("count_tumbling", 3), ("time", 2), ("time", 3)])
def test_partitioned_equals_whole_stream(oracle_lib, name, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=120) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    merged = [w for r in range(world) for w in got[r]]
    spec, g = _case(name)
    whole = gen.generate(g["kind"], g["n"], g["seed"], rate=g["rate"], groups=g["groups"])
    exp = oracle_lib.run(spec, whole)
    # the last rank's stream ends where the whole stream ends: same closed windows
    assert [w[0] for w in merged] == list(exp["win_id"])
    for k, (wid, keys, vals) in enumerate(merged):
        o, nr = exp["win_rowoff"][k], exp["win_nrows"][k]
        assert keys == [tuple(exp["keys"][r]) for r in range(o, o + nr)]
        ev = [tuple(v[r].item() for v in exp["vals"]) for r in range(o, o + nr)]
        assert vals == ev
