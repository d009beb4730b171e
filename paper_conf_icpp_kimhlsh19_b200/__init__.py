"""paper_conf_icpp_kimhlsh19_b200 — B200-native CATT hot path.

CATT (Compiler-Assisted Thread Throttling, Kim et al., ICPP 2019): a static
L1D-footprint model picks how many warps per CTA and CTAs per SM may run a
memory-divergent loop at once; hand-written sm_100a kernels enforce it.
See include/catt.h (the C ABI) and DESIGN.md.
"""
from .catt import *  # noqa: F401,F403
from . import catt  # noqa: F401

__all__ = [n for n in dir(catt) if not n.startswith("_")]
