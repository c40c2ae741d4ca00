"""B200-native brick geometric multigrid (FP64 V-cycle), after Antepara et al., SC'24.

The product is the C-ABI library ``libmg_b200.so`` (include/mg.h) built from
``csrc/`` for sm_100a; ``mg`` is its ctypes binding (same names) and
``solver`` wraps it with torch-allocated device memory and streams.
"""
from . import mg  # noqa: F401

__all__ = ["mg", "Multigrid", "LoopbackGroup"]


def __getattr__(name):
    if name in ("Multigrid", "LoopbackGroup"):
        from . import solver

        return getattr(solver, name)
    raise AttributeError(name)
