"""paper_conf_micro_wudcy12_b200 — fused relational-algebra chains (Kernel Weaver,
MICRO'12) on B200.  The product is librw.so (C ABI in include/rw.h); this package
is its thin Python binding (`rw`) plus multi-GPU orchestration (`dist`)."""
from . import rw  # noqa: F401
from .rw import Plan, RwError  # noqa: F401

__all__ = ["rw", "Plan", "RwError"]
