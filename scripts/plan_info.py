"""Print the plan-level stats (kernel kinds, grids) of every bench config (GPU)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sigmod_koliousiswfwcp16_b200 import saber
from saber_inputs import workloads
for name, (spec, g) in [("C3_G64", workloads.c3(groups=64)), ("C3_G1024", workloads.c3(groups=1024)),
                        ("C4", workloads.c4()), ("C5a", workloads.c5a()), ("C5b", workloads.c5b()),
                        ("SG1", workloads.sg1()), ("C1", workloads.c1()), ("C2", workloads.c2(sel=0.5))]:
    q = saber.Query(spec, task_bytes=1 << 30, result_mode=saber.RESULTS_DEVICE, profile=True, result_slots=8)
    st = q.stats()
    print(name, saber.SCAN_KERNELS[st["scan_kind"]], saber.WINDOW_KERNELS[st["window_kind"]],
          "scan_grid", st["scan_grid"], "window_grid", st["window_grid"], "overlap", st["overlap"], flush=True)
    q.close()
