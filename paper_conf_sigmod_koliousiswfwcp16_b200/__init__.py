"""B200-native windowed streaming-query hot path (SABER, SIGMOD'16).

The product is ``libsaber.so`` (C ABI in ``include/saber.h``; sm_100a kernels
in ``csrc/``).  ``saber`` is its thin ctypes binding and ``parallel`` the
task partitioning across GPUs (one process per GPU, halo exchange through
torch.distributed).  There is no CPU execution path.
"""
from .saber import (EAGAIN, OK, RESULTS_DEVICE, RESULTS_HOST, Query, SaberError,  # noqa: F401
                    lib, partition_plan)

__all__ = ["Query", "SaberError", "lib", "partition_plan", "RESULTS_HOST", "RESULTS_DEVICE", "OK", "EAGAIN"]
