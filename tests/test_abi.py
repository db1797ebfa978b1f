"""C-ABI boundary checks that need no GPU: the library builds, loads, exports
every function declared in include/saber.h, and refuses to run without a
device (there is no CPU fallback)."""
import ctypes as C
import os
import re

import pytest

from paper_conf_sigmod_koliousiswfwcp16_b200 import saber
from saber_inputs import workloads

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "saber.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(saber_[a-z_]+)\s*\(", src)))


def test_header_declares_expected_entry_points():
    names = _declared()
    for n in ("saber_query_create", "saber_task_submit", "saber_task_submit_device", "saber_results_poll",
              "saber_results_release", "saber_query_finish", "saber_query_destroy"):
        assert n in names


def test_library_exports_every_declared_symbol():
    L = saber.lib()
    for name in _declared():
        assert hasattr(L, name), name
    assert set(_declared()) == set(saber.SIGNATURES)   # the binding wraps exactly the header's API
    assert b"sm_100a" in L.saber_version()


def test_library_is_sm100a_cubin():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", saber.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_no_cpu_fallback_without_device():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    spec, _ = workloads.c1()
    with pytest.raises(saber.SaberError) as e:
        saber.Query(spec)
    assert e.value.status == saber.ECUDA


def test_partition_plan_count_closed_form():
    """Count-window partition planning is host arithmetic (no device needed)."""
    spec, _ = workloads.c3()
    closed, halo = saber.partition_plan(spec, 0, 0, 1 << 20)
    s, l = 32768, 1024
    assert closed == ((1 << 20) - s) // l + 1
    assert halo == closed * l
