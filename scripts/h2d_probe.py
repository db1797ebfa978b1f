"""Host-link probe (plumbing, not product): pinned H2D / D2H GB/s on this box,
and the library's host-submit ingest rate for one query (no results)."""
import time

import torch

n = 1 << 30
h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
d = torch.empty(n, dtype=torch.uint8, device="cuda")
for name, fn in (("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))):
    fn()
    torch.cuda.synchronize()
    t = time.perf_counter()
    for _ in range(5):
        fn()
    torch.cuda.synchronize()
    print(f"{name} pinned 1 GiB: {5 * n / (time.perf_counter() - t) / 1e9:.1f} GB/s")

# chunked H2D on two streams
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
torch.cuda.synchronize()
t = time.perf_counter()
for i in range(8):
    s = s1 if i % 2 == 0 else s2
    with torch.cuda.stream(s):
        d[(i % 2) * (n // 2):(i % 2 + 1) * (n // 2)].copy_(h[:n // 2], non_blocking=True)
torch.cuda.synchronize()
print(f"h2d 2 streams x 512 MiB: {8 * n / 2 / (time.perf_counter() - t) / 1e9:.1f} GB/s")

# library ingest: C3 query fed from host memory (torch-pinned vs numpy + saber_register_host)
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np
from paper_conf_sigmod_koliousiswfwcp16_b200 import saber
from saber_inputs import workloads
spec, g = workloads.c3(groups=64)
N = 8 << 30
src_t = torch.empty(N, dtype=torch.uint8, pin_memory=True)
src_n = np.zeros(N, dtype=np.uint8)
for name, arr in (("torch-pinned", src_t.numpy()), ("numpy+register", src_n)):
    for mode in (saber.RESULTS_DEVICE, saber.RESULTS_HOST):
        q = saber.Query(spec, task_bytes=1 << 30, result_mode=mode)
        t0 = time.perf_counter()
        q.register_host(arr)
        treg = time.perf_counter() - t0
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        off = 0
        while off < N:
            part = arr[off:off + (4 << 30)]
            st = q.submit(part)
            if st == saber.EAGAIN:
                st2, r = q.poll_raw(-1); q.release(r); continue
            assert st == 0, q.last_error()
            off += part.size
        while (st := q.finish()) == saber.EAGAIN:
            st2, r = q.poll_raw(-1); q.release(r)
        assert st == 0, q.last_error()
        while True:
            st2, r = q.poll_raw(-1)
            if st2 != 0: break
            q.release(r)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        print(f"{name:16s} mode={mode} register {treg:.2f}s  ingest {N / dt / 1e9:.1f} GB/s")
        q.close()
