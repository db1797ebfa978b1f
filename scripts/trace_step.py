"""Live kernel timeline of bench steps (torch.profiler / CUPTI sees every kernel of
the context, the library's too): per kernel start offset from the step's first
kernel, duration, and the idle gap before it.  1 GPU, device-resident, like bench.py.
usage: python scripts/trace_step.py [--config C3 --groups 64 --task-mb 4096 --steps 2]"""
import argparse
import ctypes as C
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_sigmod_koliousiswfwcp16_b200 import saber  # noqa: E402
from saber_inputs import gen, workloads  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3")
ap.add_argument("--groups", type=int, default=64)
ap.add_argument("--task-mb", type=int, default=0)
ap.add_argument("--steps", type=int, default=2)
ap.add_argument("--tuples-log2", type=int, default=0)
a = ap.parse_args()
fn = workloads.CONFIGS[a.config]
spec, g = fn(groups=a.groups) if a.config == "C3" else fn()
if a.tuples_log2:
    g["n"] = 1 << a.tuples_log2
tb = spec["schema"]["tuple_bytes"]
lib_gen = C.CDLL(os.path.join(ROOT, "saber_inputs", "libsaber_gen.so"))
part = torch.empty(g["n"] * tb, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream()
assert lib_gen.saber_gen(gen.KIND_ID[g["kind"]], C.c_uint64(g["seed"]), C.c_int64(0), C.c_int64(g["n"]),
                         C.c_int64(g.get("rate", 1)), C.c_int64(g.get("groups", 64)), C.c_void_p(part.data_ptr()),
                         C.c_void_p(s.cuda_stream)) == 0
torch.cuda.synchronize()
task = (a.task_mb or workloads.bench_task_mb(a.config, a.groups)) << 20
q = saber.Query(spec, task_bytes=task, result_mode=saber.RESULTS_DEVICE, result_slots=8)
tt = q.stats()["task_tuples"] * tb


import time  # noqa: E402
HT = []


def step():
    q.reset(0, 0)
    torch.cuda.synchronize()
    off = 0
    while off < part.numel():
        nb = min(tt, part.numel() - off)
        t0 = time.perf_counter()
        st = q.submit_device(part.data_ptr() + off, nb, s.cuda_stream)
        HT.append(("submit", (time.perf_counter() - t0) * 1e6))
        if st == saber.EAGAIN:
            st_, r = q.poll_raw(-1)
            if st_ == 0:
                q.release(r)
            continue
        assert st == 0, q.last_error()
        off += nb
    t0 = time.perf_counter()
    while q.finish() == saber.EAGAIN:
        st_, r = q.poll_raw(-1)
        if st_ == 0:
            q.release(r)
    HT.append(("finish", (time.perf_counter() - t0) * 1e6))
    q.record(s.cuda_stream)
    while q.stats()["tasks_pending"] > 0:
        st_, r = q.poll_raw(-1)
        if st_ == 0:
            q.release(r)
    torch.cuda.synchronize()


for _ in range(3):
    step()
from torch.profiler import ProfilerActivity, profile  # noqa: E402

with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
    for _ in range(a.steps):
        step()
ev = [e for e in prof.events() if e.device_type.name == "CUDA"]
ev.sort(key=lambda e: e.time_range.start)
t0 = ev[0].time_range.start if ev else 0
prev_end = t0
for e in ev:
    st, en = e.time_range.start, e.time_range.end
    print(f"{(st - t0):10.1f} us  dur {en - st:9.1f}  gap {st - prev_end:7.1f}  {e.name[:70]}")
    prev_end = max(prev_end, en)
print('host us:', [(a, round(b, 1)) for a, b in HT[-6:]])
q.close()
