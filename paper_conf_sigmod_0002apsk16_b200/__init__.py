"""B200-native GTS hot path (Kim et al., SIGMOD'16): slotted-page BFS, PageRank,
SSSP and WCC as hand-written sm_100a CUDA kernels behind a C ABI (libgts.so,
include/gts.h).  This package is only the thin ctypes binding (gts.py)."""
from .gts import *  # noqa: F401,F403
from .gts import EXPORTED, GtsError, Graph, Context  # noqa: F401
