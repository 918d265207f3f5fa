"""B200-native variable-size batched LU / TRSV / block-Jacobi (sm_100a).

Hot path of Anzt, Dongarra, Flegar, Quintana-Orti (ICPP 2017) behind the C
ABI in ``include/bj.h``; ``bj`` is the ctypes binding.  See DESIGN.md.
"""
from . import bj  # noqa: F401

__all__ = ["bj"]
