"""CPU oracle for Neo's Hybrid key-switching hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / ``--impl reference``
legs may import, call, link or execute anything under oracle/.  The product path
(paper_conf_isca_jiaodwfcm0z25_b200) never does, and fails loudly without its CUDA
library.  See oracle/ckks.py for what is computed and the paper passages it follows.
"""
from ._core import build  # noqa: F401
