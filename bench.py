#!/usr/bin/env python
"""Benchmark: one windowed query over a synthetic stream on 1..8 B200s.

Default workload (BASELINE.json configs[2], SURVEY.md §8 "C3"): Syn 32-byte
tuples, ``SELECT AVG(a1) FROM Syn [ROWS 32768 SLIDE 1024] GROUP BY a2`` with
G = 64 groups, 2^28 tuples (8 GiB) per GPU.  A step is one pass of the whole
hot path -- task dispatch, K1 boundary/pane assignment + σ + pane partial
aggregation, window assembly and the result stage -- over the GPU's stream
partition (plus the halo exchange when N > 1).  Multi-GPU is weak scaling:
rank r owns tuples [r·2^28, (r+1)·2^28) of one global stream of N·2^28 tuples
and emits the windows closed inside its partition; only the halo (< s tuples)
crosses NVLink, once per step.

``value``  tuples/s, device-resident (inputs already in HBM), whole job / max rank time
``e2e``    the same metric through the C ABI from pinned HOST buffers, H2D of the
           inputs and D2H of every result slice inside the timed region
``--impl reference``  the CPU oracle (oracle/) timed on this host's cores on a
           bounded sample of the same workload (the reference arm of this tier)
"""
from __future__ import annotations

import argparse
import ctypes as C
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from saber_inputs import gen, workloads  # noqa: E402

METRIC = "tuples/s & GB/s per windowed query at 1/2/4/8 B200; % of HBM roofline"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="saber", choices=["saber", "reference"])
    ap.add_argument("--config", default="C3", choices=["C1", "C2", "C3", "C4", "C5a", "C5b", "SG1", "CM2", "JOIN"])
    ap.add_argument("--join-r", type=int, default=4, help="JOIN: predicates r of JOIN_r (Table 1, L1385)")
    ap.add_argument("--npred", type=int, default=1,
                    help="C2: SELECT_n -- n predicate terms (n-1 always-true terms, Fig. 10a)")
    ap.add_argument("--groups", type=int, default=64)
    ap.add_argument("--sel", type=float, default=0.5)
    ap.add_argument("--rate", type=int, default=0)
    ap.add_argument("--tuples-log2", type=int, default=0, help="tuples per GPU (default: the config's)")
    ap.add_argument("--task-mb", type=int, default=0,
                    help="query task size φ in MiB (device-resident leg; default: the config's, "
                         "saber_inputs.workloads.BENCH_TASK_MB -- B200 plateau: DESIGN.md §8 φ sweep)")
    ap.add_argument("--e2e-task-mb", type=int, default=256,
                    help="task size φ of the end-to-end leg (finer tasks pipeline H2D with compute)")
    ap.add_argument("--size", type=int, default=0, help="override the window size (slide sweeps, Fig. 11)")
    ap.add_argument("--slide", type=int, default=0, help="override the window slide (slide sweeps, Fig. 11)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--hash-capacity", type=int, default=0,
                    help="pane hash-table slots (power of two; 0: the planner's guess).  CM2 defaults to "
                         "2x the expected distinct jobIds per pane (the paper's static hash-table pool, L1293-1295)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo: multi-rank plumbing check with ranks sharing GPUs (collectives via the host)")
    ap.add_argument("--launcher-check", action="store_true",
                    help="CPU (gloo) check of the multi-rank launch: no GPU work")
    return ap.parse_args()


def workload(args):
    c = args.config
    if c == "C1":
        spec, g = workloads.c1()
    elif c == "C2":
        spec, g = workloads.c2(sel=args.sel, npred=args.npred)
    elif c == "C3":
        spec, g = workloads.c3(groups=args.groups)
    elif c == "C4":
        spec, g = workloads.c4(rate=args.rate or 64)
    elif c == "C5a":
        spec, g = workloads.c5a(rate=args.rate or 4096)
    elif c == "C5b":
        spec, g = workloads.c5b(rate=args.rate or 8192)
    elif c == "CM2":
        spec, g = workloads.cm2(rate=args.rate or 64)
    else:
        spec, g = workloads.sg1(rate=args.rate or 4096)
    if args.tuples_log2:
        g["n"] = 1 << args.tuples_log2
    w = spec["window"]
    if args.size:
        w["size"] = args.size
    if args.slide:
        w["slide"] = args.slide
    desc = {
        "C1": "Syn 32-B, SUM(a1), count w(1024,1024)",
        "C2": f"Syn 32-B, SELECT ts,a1,a2 WHERE a3<sel*2^31 (sel={args.sel}), count w(1024,64), IStream",
        "C3": f"Syn 32-B, AVG(a1) GROUP BY a2 (G={args.groups}), count w(32768,1024)",
        "C4": f"CM 64-B, SUM(cpu) GROUP BY category, time w(60,1), R={g['rate']}/s",
        "C5a": f"SG 32-B, AVG(value) GROUP BY plug,household,house, time w(3600,1), R={g['rate']}/s",
        "C5b": f"LRB 32-B, AVG(speed) GROUP BY highway,direction,position/5280 HAVING avg<40, time w(300,1), R={g['rate']}/s",
        "SG1": f"SG 32-B, AVG(value), time w(3600,1), R={g['rate']}/s",
        "CM2": f"CM 64-B, AVG(cpu) WHERE eventType==1 GROUP BY jobId (int64, undeclared), time w(60,1), R={g['rate']}/s",
    }[c]
    if c == "C2" and args.npred > 1:
        desc += f" [SELECT_{args.npred}: {args.npred - 1} extra always-true terms]"
    if args.size or args.slide:
        desc += f" [window overridden: size {w['size']}, slide {w['slide']}]"
    name = f"{c}: {desc}, 2^{int(np.log2(g['n']))} tuples ({g['n'] * spec['schema']['tuple_bytes'] >> 20} MiB) per GPU"
    return spec, g, name, w


# --------------------------------------------------------------------------- utils
class Clocks:
    """SM clocks and clock-event reasons sampled DURING the timed region (the
    recipe's clocks line).  NVML is polled every ~2 ms from a thread (the timed
    region of a step is milliseconds, too short for `nvidia-smi -lms`); samples
    are tagged with whether a timed step was in flight (``clk.timed = True``).
    Every sample is also written to ``path`` as CSV."""

    REASONS = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
               "hw_power_brake_slowdown": 0x80, "sw_power_cap": 0x4}

    def __init__(self, index, path):
        self.index, self.path = index, path
        self.rows, self.timed, self._stop = [], False, False
        self.thread = None
        self.error = None

    def _run(self):
        import pynvml
        for attempt in range(20):                   # NVML init can fail transiently right after another process
            try:
                pynvml.nvmlInit()
                break
            except Exception as e:                  # noqa: BLE001
                self.error = f"nvmlInit: {e}"
                time.sleep(0.05)
        else:
            return
        try:
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            reasons = getattr(pynvml, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
                pynvml.nvmlDeviceGetCurrentClocksThrottleReasons
            while not self._stop:
                sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                rs = reasons(h)
                self.rows.append((time.perf_counter(), self.timed, sm, mx, int(rs)))
                time.sleep(0.002)
        except Exception as e:                      # noqa: BLE001
            self.error = f"nvml: {e}"
        finally:
            pynvml.nvmlShutdown()

    def smi_once(self):
        """Fallback when NVML sampling produced nothing: one nvidia-smi reading."""
        try:
            out = subprocess.run(["nvidia-smi", "-i", str(self.index), "--query-gpu=clocks.sm,clocks.max.sm,"
                                  "clocks_event_reasons.active", "--format=csv,noheader,nounits"],
                                 capture_output=True, text=True, timeout=20).stdout.strip().split(",")
            return int(out[0]), int(out[1]), int(out[2].strip(), 16)
        except Exception:                           # noqa: BLE001
            return None

    def __enter__(self):
        try:
            import pynvml  # noqa: F401
            self.thread = threading.Thread(target=self._run, daemon=True)
            self.thread.start()
        except Exception:
            self.thread = None
        return self

    def __exit__(self, *a):
        self._stop = True
        if self.thread:
            self.thread.join(timeout=5)
        try:
            with open(self.path, "w") as f:
                f.write("t,timed,sm_mhz,sm_max_mhz,reasons\n")
                for r in self.rows:
                    f.write(f"{r[0]:.6f},{int(r[1])},{r[2]},{r[3]},{r[4]:#x}\n")
        except Exception:
            pass

    def summary(self):
        rows = [r for r in self.rows if r[1]]
        where = "timed region"
        if not rows:
            rows, where = self.rows, "whole run (no sample fell inside a timed step)"
        if not rows:
            one = self.smi_once()
            if one is None:
                return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0,
                        "error": self.error}
            rows, where = [(0.0, False, one[0], one[1], one[2])], "after the timed region (nvidia-smi, NVML failed)"
        reasons = sorted({n for r in rows for n, bit in self.REASONS.items() if r[4] & bit})
        return {"sm_mhz": statistics.median(r[2] for r in rows), "sm_max_mhz": max(r[3] for r in rows),
                "reasons": reasons, "samples": len(rows), "sampled": where,
                "source": "nvidia-smi" if where.startswith("after") else "NVML, ~2 ms poll"}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def host_link(dev, nbytes=256 << 20, reps=10):
    """Pinned host<->device copy bandwidth of this GPU, measured in the same run
    (SURVEY.md §8(d) D5): best of `reps` cudaMemcpyAsync of 256 MiB each way."""
    import torch
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    out = {}
    for name, dst, src in (("h2d_gbs", d, h), ("d2h_gbs", h, d)):
        best = None
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            dst.copy_(src, non_blocking=True)
            e1.record()
            e1.synchronize()
            ms = e0.elapsed_time(e1)
            best = ms if best is None else min(best, ms)
        out[name] = nbytes / (best / 1e3) / 1e9
    del h, d
    return out


def ncu_traffic(config_key):
    """Per-launch DRAM bytes of the dominant kernel from a committed ncu --set full capture."""
    path = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return d.get(config_key)
    except Exception:
        return None


def gen_device(lib_gen, kind, seed, i0, n, rate, groups, out, stream):
    rc = lib_gen.saber_gen(gen.KIND_ID[kind], C.c_uint64(seed), C.c_int64(i0), C.c_int64(n), C.c_int64(rate),
                           C.c_int64(groups), C.c_void_p(out.data_ptr()), C.c_void_p(stream))
    assert rc == 0, rc


# --------------------------------------------------------------------------- reference arm
def cpu_oracle_sample(spec, g, budget_s, threads):
    """Time the oracle (as it stands) on a bounded prefix of the same workload.
    Returns (tuples/s of stream covered, sample description)."""
    import oracle
    oracle.build()
    w = spec["window"]
    tb = spec["schema"]["tuple_bytes"]
    rate = g.get("rate", 1)
    unit = w["slide"] if w["kind"] == "count" else w["slide"] * rate     # tuples per window step

    def run(nw):
        if w["kind"] == "count":
            ntup = (nw - 1) * w["slide"] + w["size"]
        else:
            ntup = ((nw - 1) * w["slide"] + w["size"] + 1) * rate
        data = gen.generate(g["kind"], ntup, g["seed"], rate=rate, groups=g["groups"])
        t0 = time.perf_counter()
        r = oracle.run(spec, data, windows=list(range(nw)), nthreads=threads)
        dt = time.perf_counter() - t0
        assert len(r["win_id"]) == nw
        return dt, ntup

    nw = 16
    dt, _ = run(nw)
    while dt < 0.5 and nw < (1 << 22):
        nw *= 4
        dt, _ = run(nw)
    nw = max(16, int(nw * budget_s / max(dt, 1e-3)))
    dt, ntup = run(nw)
    value = nw * unit / dt
    sample = (f"first {nw} windows of the workload's stream ({ntup} tuples read, {nw * unit} tuples of stream "
              f"advanced), oracle recomputes every window from scratch; value = stream tuples advanced / wall s")
    return value, sample, dt


def run_config(args, spec, g, name, world):
    """The workload's static description, identical for both arms (--impl saber /
    reference); run-dependent counters are reported outside it."""
    tb = spec["schema"]["tuple_bytes"]
    n = g["n"]
    return {"workload": name, "groups": args.groups if args.config == "C3" else None,
            "task_bytes": (args.task_mb or workloads.bench_task_mb(args.config, args.groups)) << 20,
            "tuples_per_gpu": n,
            "l2": ("flushed: a 512 MiB memset before every step (input < 2x the 126 MB L2)"
                   if n * tb < (256 << 20) else
                   f"inputs ({n * tb >> 20} MiB per GPU) exceed the 126 MB L2: no flush needed"),
            "parallelism": f"dp{world} (stream partitions + halo)"}


def run_reference(args, spec, g, name, rank, world):
    if rank != 0:
        return
    threads = len(os.sched_getaffinity(0))
    vals = []
    for i in range(args.warmup + args.steps):
        v, sample, dt = cpu_oracle_sample(spec, g, max(2.0, args.cpu_seconds / max(1, args.steps)), threads)
        if i >= args.warmup:
            vals.append(v)
    value = statistics.median(vals)
    line = {"metric": METRIC, "value": value, "unit": "tuples/s", "impl": "reference", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": None, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": run_config(args, spec, g, name, world),
            "cpu_baseline": {"value": value, "unit": "tuples/s", "cores": threads, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": value, "unit": "tuples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------------- product arm
def launch_ranks(n):
    """``--gpus N`` outside a torchrun environment: start N ranks, one process per
    GPU, through torch.distributed.run on 127.0.0.1, and return its exit code
    (rank 0 prints the JSON line).  Inside torchrun, WORLD_SIZE must equal N."""
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def launcher_check(args, rank, world):
    """CPU check of the multi-rank plumbing (gloo): rendezvous, world size, the
    max-over-ranks reduction of step times and rank-0-only output."""
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo")
    t = torch.tensor([float(rank + 1)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if rank == 0:
        print(json.dumps({"launcher_check": True, "n_gpus": world, "ms_max": float(t.item()),
                          "ranks": dist.get_world_size()}), flush=True)
    dist.destroy_process_group()


def run_join(args, rank, world):
    """f3: JOIN_r over two Syn streams of 2^tuples_log2 tuples each (default 2^20),
    ω(size, slide) (default the paper's ω32KB,32KB = 1024 tuples), device-resident
    batches of φ tuples, DEVICE results.  Value: input tuples (both streams) / s.
    The join is ALU-bound: s^2 pair tests per window; roofline.bound = "alu" with
    the pair-test rate against a peak derived in DESIGN.md §6."""
    import torch
    from paper_conf_sigmod_koliousiswfwcp16_b200 import saber
    size = args.size or 1024
    slide = args.slide or size
    n = 1 << (args.tuples_log2 or 20)
    js, g = workloads.join_r(r=args.join_r, size=size, slide=slide, n=n)
    name = (f"JOIN_{args.join_r}: Syn x Syn, theta = {args.join_r} terms S1.a_k < S2.a_k, count w({size},{slide}), "
            f"2^{int(np.log2(n))} tuples per stream")
    dev = torch.device("cuda", 0)
    lib_gen = C.CDLL(os.path.join(ROOT, "saber_inputs", "libsaber_gen.so"))
    st = torch.cuda.current_stream()
    bufs = []
    for seed in (g["seed1"], g["seed2"]):
        b = torch.empty(n * 32, dtype=torch.uint8, device=dev)
        gen_device(lib_gen, "syn", seed, 0, n, 1, 64, b, st.cuda_stream)
        bufs.append(b)
    torch.cuda.synchronize()
    # tasks of 4 MiB per stream by default: a task's pair rows (selectivity 2^-min(r, 4) of
    # s^2 per window, 16 B each) must fit its result slot, sized from that estimate
    batch = max(size, ((args.task_mb or 4) << 20) // 32)
    batch = min(batch, n)
    nt = (n + batch - 1) // batch
    est_pairs = (batch // slide + 1) * size * size / 2 ** min(args.join_r, 4)
    rbytes = int(min(8 << 30, max(64 << 20, est_pairs * 16 * 1.25)))
    j = saber.Join(js, task_bytes=batch * 32, result_mode=saber.RESULTS_DEVICE, result_slots=nt + 1,
                   result_bytes=rbytes)
    times, pairs = [], 0
    with Clocks(0, os.path.join(ROOT, "gpurun_out", "clocks_join.csv") if os.path.isdir(os.path.join(ROOT, "gpurun_out"))
                else "/tmp/clocks_join.csv") as clk:
        for it in range(args.warmup + args.steps):
            j.close()
            j = saber.Join(js, task_bytes=batch * 32, result_mode=saber.RESULTS_DEVICE, result_slots=nt + 1,
                           result_bytes=rbytes)
            torch.cuda.synchronize()
            clk.timed = it >= args.warmup
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            for t in range(nt):
                k = min(batch, n - t * batch)
                rc = j.submit_device(bufs[0].data_ptr() + t * batch * 32, bufs[1].data_ptr() + t * batch * 32, k,
                                     st.cuda_stream)
                assert rc == 0, j.last_error()
            e1.record(st)
            torch.cuda.synchronize()
            clk.timed = False
            tot = 0
            for _ in range(nt):
                rc, r = j.poll_raw(-1)
                if rc != 0:                    # e.g. ENOMEM: the pairs did not fit a slot -- never a bench value
                    raise saber.SaberError(rc, j.last_error())
                tot += r.ntuples
                j.release(r)
            if it >= args.warmup:
                times.append(e0.elapsed_time(e1))
                pairs = tot
    j.close()
    ms = statistics.median(times)
    nwin = (n - size) // slide + 1
    tests = nwin * size * size
    tests_per_s = tests / (ms / 1e3)
    # two bounds: ALU -- a pair test needs at least a compare and a select
    # per θ term on one INT32 lane (B200: 148 SMs x 128 INT32 lanes per clock); HBM -- the
    # pair rows written.  The roofline reports the binding one (the larger time)
    clk_ghz = MEASURED_SM_GHZ
    peak = 148 * 128 * clk_ghz * 1e9 / (2 * args.join_r)
    ctype = {c[0]: c[1] for c in js["schema1"]["cols"]} if "schema1" in js else {}
    row_bytes = sum(8 if ctype.get(c, "i32") in ("i64", "f64") else 4 for c in js.get("project1", [])) + \
        4 * len(js.get("project2", []))          # JOIN_r: S1.ts (8) + S1.a1 + S2.a1 + S2.a2 = 20 B
    hbm_peak, hbm_src = measured_peaks()
    t_alu = tests / peak
    t_hbm = pairs * row_bytes / (hbm_peak * 1e9)
    line = {"metric": METRIC, "value": 2 * n / (ms / 1e3), "unit": "tuples/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "i32", "data": "synthetic",
            "config": {"workload": name, "task_tuples": batch, "windows_per_step": nwin, "pairs_out_per_step": pairs},
            "roofline": ({"bound": "alu", "achieved": tests_per_s, "peak": peak, "unit": "pair tests/s",
                          "frac": tests_per_s / peak,
                          "peak_source": "derived: 148 SMs x 128 INT32 lanes x SM clock / (2 instructions x r terms "
                                         "per pair test)"} if t_alu >= t_hbm else
                         {"bound": "hbm", "achieved": pairs * row_bytes / (ms / 1e3) / 1e9, "peak": hbm_peak,
                          "unit": "GB/s", "frac": pairs * row_bytes / (ms / 1e3) / 1e9 / hbm_peak,
                          "peak_source": hbm_src, "note": f"pair rows written ({row_bytes} B each)"}) |
                        {"pair_tests_per_s": tests_per_s, "alu_bound_ms": t_alu * 1e3, "hbm_bound_ms": t_hbm * 1e3},
            "clocks": clk.summary(), "gpu_launches": 5 * nt}
    if rank == 0:
        print(json.dumps(line), flush=True)


MEASURED_SM_GHZ = 1.965


def main():
    args = parse()
    if args.config == "JOIN":
        run_join(args, int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")))
        return
    spec, g, name, w = workload(args)
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        sys.exit(launch_ranks(args.gpus))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.dist_backend == "gloo":
        # plumbing check of the multi-rank path on a box with fewer GPUs than ranks:
        # ranks share the visible GPUs round-robin, collectives go through the host
        import torch
        local = local % max(1, torch.cuda.device_count())
    if world != args.gpus:
        print(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}", file=sys.stderr)
        sys.exit(2)
    if args.launcher_check:
        launcher_check(args, rank, world)
        return
    import torch
    import torch.distributed as dist
    if world > 1:
        torch.cuda.set_device(local)
        if args.dist_backend == "gloo":
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    if args.impl == "reference":
        run_reference(args, spec, g, name, rank, world)
        if world > 1:
            dist.destroy_process_group()
        return

    from paper_conf_sigmod_koliousiswfwcp16_b200 import saber
    from paper_conf_sigmod_koliousiswfwcp16_b200.parallel import exchange_halo
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    lib_gen = C.CDLL(os.path.join(ROOT, "saber_inputs", "libsaber_gen.so"))
    tb = spec["schema"]["tuple_bytes"]
    n = g["n"]                                   # tuples per GPU (weak scaling)
    begin = rank * n
    part = torch.empty(n * tb, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()
    gen_device(lib_gen, g["kind"], g["seed"], begin, n, g["rate"], g["groups"], part, stream.cuda_stream)
    torch.cuda.synchronize()
    task_bytes = (args.task_mb or workloads.bench_task_mb(args.config, args.groups)) << 20

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev if args.dist_backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def drive(q, pieces, s):
        """Submit device pieces (ptr, nbytes) in task-sized chunks; poll+release
        whenever all result slots are busy.  Returns (windows, rows, tuples out)."""
        nw = nr = nt = 0

        def drain_one():
            nonlocal nw, nr, nt
            st, r = q.poll_raw(-1)
            if st != 0:
                raise saber.SaberError(st, q.last_error())
            nw += r.nwindows; nr += r.nrows; nt += r.ntuples
            q.release(r)
        for ptr, nbytes in pieces:
            off = 0
            while off < nbytes:
                nb = min(task_bytes, nbytes - off)
                st = q.submit_device(ptr + off, nb, s)
                if st == saber.EAGAIN:
                    drain_one()
                    continue
                if st != 0:
                    raise saber.SaberError(st, q.last_error())
                off += nb
        while (st := q.finish()) == saber.EAGAIN:
            drain_one()
        if st != 0:
            raise saber.SaberError(st, q.last_error())
        q.record(s)
        return drain_one, (lambda: (nw, nr, nt))

    # ---------------- device-resident timed loop
    # partition planning metadata (first window / base index) is fixed by the data;
    # the query objects are created outside the timed region, the halo bytes are
    # exchanged inside it every step.
    def halo_exchange():
        if args.dist_backend == "nccl":
            return exchange_halo(spec, part, begin, n, rank, world)
        # gloo (plumbing check, small partitions): the window arithmetic on the device
        # (saber_partition_plan), the bytes through the host
        from paper_conf_sigmod_koliousiswfwcp16_b200.saber import partition_plan
        h, fw, bi = exchange_halo(spec, part.cpu(), begin, n, rank, world,
                                  plan=lambda sp, pt, b, m: partition_plan(sp, part.data_ptr(), b, m))
        return h.to(dev), fw, bi

    if world > 1:
        _, first_window, base_index = halo_exchange()
    else:
        first_window, base_index = 0, begin
    times, stats_acc = [], []
    out_rows = out_tuples = out_windows = 0
    clk_dir = os.path.join(ROOT, "gpurun_out") if os.path.isdir(os.path.join(ROOT, "gpurun_out")) else "/tmp"
    # one long-lived query; every step replays the stream after saber_query_reset
    hcap = args.hash_capacity
    if not hcap and args.config == "CM2":
        # eventType == 1 keeps 1/9 of R tuples per 1-s pane; their jobIds are ~all distinct
        hcap = 1 << max(6, int(np.ceil(np.log2(2 * max(1, g["rate"] // 9)))))
    q = saber.Query(spec, base_index=base_index, first_window=first_window,
                    emit_on_finish=(rank == world - 1), task_bytes=task_bytes,
                    result_mode=saber.RESULTS_DEVICE, profile=True, result_slots=8, device=local,
                    hash_capacity=hcap)
    with Clocks(local, os.path.join(clk_dir, f"clocks_rank{rank}.csv")) as clk:
        t_wait = time.perf_counter()                 # NVML initialised and sampling before timing
        while clk.thread is not None and not clk.rows and time.perf_counter() - t_wait < 5.0:
            time.sleep(0.01)
        # inputs smaller than twice the 126 MB L2 (C1: 32 MiB) would be re-read from L2
        # across steps: every step then starts behind a 512 MiB memset (outside the timed region)
        l2_flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev) if n * tb < (256 << 20) else None
        for it in range(args.warmup + args.steps):
            q.reset(base_index, first_window)
            if l2_flush is not None:
                l2_flush.zero_()
            barrier()
            torch.cuda.synchronize()
            ev0 = torch.cuda.Event(enable_timing=True)
            ev1 = torch.cuda.Event(enable_timing=True)
            clk.timed = it >= args.warmup
            ev0.record(stream)
            pieces = []
            if world > 1:
                halo, fw, bi = halo_exchange()
                assert (fw, bi) == (first_window, base_index)
                if halo.numel():
                    pieces.append((halo.data_ptr(), halo.numel()))
            pieces.append((part.data_ptr(), part.numel()))
            drain_one, counts = drive(q, pieces, stream.cuda_stream)
            ev1.record(stream)
            while q.stats()["tasks_pending"] > 0:     # already complete once ev1 is
                drain_one()
            torch.cuda.synchronize()
            clk.timed = False
            ms = ev0.elapsed_time(ev1)
            st = q.stats()
            if it >= args.warmup:
                times.append(ms)
                stats_acc.append(st)
                out_windows, out_rows, out_tuples = counts()
    q.close()
    clocks = clk.summary()
    ms_rank = statistics.median(times)
    print(f"[bench rank {rank}] device-resident step ms: {[round(t, 3) for t in times]}", file=sys.stderr)
    ms_step = max_over_ranks(ms_rank)
    total_tuples = n * world
    value = total_tuples / (ms_step / 1e3)

    # roofline of the dominant kernel (the fused K1+σ+pane-aggregation scan, or K1+K3 for σ/π)
    scan_ms = sum(s["scan_ms"] for s in stats_acc)
    scan_launches = sum(s["scan_launches"] for s in stats_acc)
    launches = sum(s["kernel_launches"] for s in stats_acc)
    bytes_scanned = sum(s["bytes_in"] for s in stats_acc)        # 1 x 32-B sector per 32-B tuple read
    peak, peak_src = measured_peaks()
    per_launch_bytes = bytes_scanned / max(1, scan_launches)
    per_launch_ms = scan_ms / max(1, scan_launches)
    achieved = per_launch_bytes / (per_launch_ms / 1e3) / 1e9 if per_launch_ms > 0 else None
    key = f"{args.config}_G{args.groups}" if args.config == "C3" else args.config
    traffic, traffic_note = ncu_traffic(key), None
    if isinstance(traffic, dict):
        cap_in = traffic["launch_input_bytes"]
        traffic = traffic["dram_bytes"] * (per_launch_bytes / cap_in) if cap_in else None
        if cap_in != int(per_launch_bytes):
            traffic_note = f"scaled from an ncu capture of a {cap_in >> 20} MiB launch"
    # whole-step roofline: algorithmic bytes of the step (input sectors read + result
    # rows, headers and projected tuples written) / step time
    ctype = {c[0]: c[1] for c in spec["schema"]["cols"]}
    row_bytes = sum(4 if ctype[c] == "i32" else 8 for c, _, _ in spec.get("group_by", [])) + 8 * len(spec.get("aggs", []))
    proj_bytes = sum(4 if ctype[c] in ("i32", "f32") else 8 for c in spec.get("project", []))
    step_bytes = n * tb + out_rows * row_bytes + out_windows * 32 + out_tuples * proj_bytes   # per GPU
    step_gbs = step_bytes / (ms_step / 1e3) / 1e9
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": (achieved / peak) if achieved else None,
                "step_achieved": step_gbs, "step_frac": step_gbs / peak, "step_bytes_per_gpu": step_bytes,
                "traffic": traffic, "traffic_note": traffic_note,
                "kernel": saber.SCAN_KERNELS[stats_acc[-1]["scan_kind"]] if stats_acc else None,
                "window_kernels": saber.WINDOW_KERNELS[stats_acc[-1]["window_kind"]] if stats_acc else None,
                "algorithmic_bytes_per_launch": per_launch_bytes, "avg_launch_ms": per_launch_ms,
                "launches_per_step": scan_launches / max(1, len(stats_acc)), "peak_source": peak_src,
                "scan_grid": stats_acc[-1]["scan_grid"] if stats_acc else None,
                "window_grid": stats_acc[-1]["window_grid"] if stats_acc else None,
                "share_of_step": (scan_ms / max(1, len(stats_acc))) / ms_rank if ms_rank else None,
                "window_ms_per_step": sum(s["assemble_ms"] for s in stats_acc) / max(1, len(stats_acc)),
                "overlap": bool(stats_acc[-1]["overlap"]) if stats_acc else None}

    # ---------------- end-to-end through the C ABI from pinned host memory
    e2e = None
    if not args.no_e2e:
        host = torch.empty(n * tb, dtype=torch.uint8, pin_memory=True)
        host.copy_(part)
        torch.cuda.synchronize()
        host_np = host.numpy()
        e_times = []
        d2h_bytes = 0
        e2e_task = args.e2e_task_mb << 20
        q = saber.Query(spec, task_bytes=e2e_task, result_mode=saber.RESULTS_HOST, device=local,
                        base_index=base_index, first_window=first_window, emit_on_finish=(rank == world - 1),
                        hash_capacity=hcap)
        q.register_host(host_np)
        for it in range(args.warmup + min(args.steps, 3)):
            q.reset(base_index, first_window)
            barrier()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            halo_np = None
            if world > 1:
                halo, _, _ = halo_exchange()
                halo_np = halo.cpu().numpy() if halo.numel() else None
            got_bytes = 0
            chunks = []
            if halo_np is not None:
                chunks.append(halo_np)
            chunks.append(host_np)
            per = e2e_task * 7

            def take():
                """Next result slice through the C ABI: poll returns once the slice's
                headers and rows are in the query's pinned host mirror (the D2H read
                of the result); count its bytes and hand the slot back."""
                st, r = q.poll_raw(-1)
                if st != 0:
                    raise saber.SaberError(st, q.last_error())
                nb = r.nrows * sum(r.col_bytes[c] for c in range(r.ncols)) + r.ntuples * r.tuple_bytes + \
                    (r.nwindows * 32 if r.hdr else 0)
                q.release(r)
                return nb
            for arr in chunks:
                off = 0
                while off < arr.size:
                    part_np = arr[off:off + per]
                    st = q.submit(part_np)
                    if st == saber.EAGAIN:
                        got_bytes += take()
                        continue
                    if st != 0:
                        raise saber.SaberError(st, q.last_error())
                    off += part_np.size
            while (st := q.finish()) == saber.EAGAIN:
                got_bytes += take()
            if st != 0:
                raise saber.SaberError(st, q.last_error())
            while q.stats()["tasks_pending"] > 0:
                got_bytes += take()
            torch.cuda.synchronize()
            dt = time.perf_counter() - t0
            if it >= args.warmup:
                e_times.append(dt)
                d2h_bytes = got_bytes
        q.close()
        e_s = max_over_ranks(statistics.median(e_times))
        link = host_link(dev)
        in_gbs = n * tb / e_s / 1e9                          # per GPU
        e2e = {"value": total_tuples / e_s, "unit": "tuples/s", "h2d_bytes_per_step": n * tb,
               "d2h_bytes_per_step": d2h_bytes, "s_per_step": e_s, "task_bytes": e2e_task,
               "input_gbs": total_tuples * tb / e_s / 1e9,
               "host_link": {"bound": "h2d", "achieved": in_gbs, "peak": link["h2d_gbs"], "unit": "GB/s",
                             "frac": in_gbs / link["h2d_gbs"], "d2h_peak": link["d2h_gbs"],
                             "peak_source": "measured in this run: pinned cudaMemcpyAsync of 256 MiB, best of 10, per GPU"}}

    # ---------------- CPU oracle baseline (rank 0, N = 1)
    cpu = None
    if not args.no_cpu and world == 1 and rank == 0:
        threads = len(os.sched_getaffinity(0))
        v, sample, dt = cpu_oracle_sample(spec, g, args.cpu_seconds, threads)
        cpu = {"value": v, "unit": "tuples/s", "cores": threads, "kind": "oracle", "sample": sample,
               "seconds": dt}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "tuples/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "f64", "data": "synthetic",
                "input_gbs": total_tuples * tb / (ms_step / 1e3) / 1e9,
                "config": run_config(args, spec, g, name, world),
                "output_per_step": {"windows": out_windows, "rows": out_rows, "out_tuples": out_tuples},
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
                "gpu_launches": launches}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
