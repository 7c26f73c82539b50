"""B200-native CA-GMRES(s, m) hot path (Yamazaki et al., IPDPS 2014).

The compute path is libcagmres.so (hand-written sm_100a FP64 kernels + NCCL); this package
is its thin Python binding.  See include/cagmres.h and DESIGN.md.
"""
from ._lib import CagmresError, load  # noqa: F401


def __getattr__(name):
    if name == "Solver":
        from .solver import Solver
        return Solver
    if name == "Plan":
        from .host import Plan
        return Plan
    raise AttributeError(name)
