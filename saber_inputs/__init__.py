"""Seeded, synthetic inputs shared by the oracle side and the CUDA side.

This package holds NO arithmetic of the method (no windows, panes, predicates
or aggregates).  It only produces:

* byte streams of row-major tuples shaped like the paper's workloads
  (``gen``: Syn / CM / SG / LRB, PAPER.md L1473-1498 and
  App. A), from a counter-based generator so the same bytes can be
  produced on the host (numpy) and on the device (``csrc/gen.cu``);
* query *specifications* as plain dicts (``workloads``): the text of a
  query, not an evaluation of it.  Each side (``oracle/`` and the product
  binding) has its own marshaller from these dicts.
"""
from . import gen, workloads  # noqa: F401
