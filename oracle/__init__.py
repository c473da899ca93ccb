"""Buffalo CPU ORACLE — test infrastructure only.

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s `cpu_baseline` / `--impl reference`
legs may import this package.  The product path (paper_conf_hpca_yangzl25_b200) never
imports it and shares no code with it.  See oracle/core.py for the per-function citations
and DESIGN.md ("Oracle", "Readings") for the paper passages each function follows.
"""
from .core import *  # noqa: F401,F403
