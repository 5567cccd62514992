"""B200-native NPB-EP hot path of the HPL paper (Bozkus & Fraguela, IPDPSW'12).

The product is the C-ABI library ``libhpl.so`` (include/hpl.h) built from
``csrc/`` for sm_100a; :mod:`.hpl` is its thin ctypes binding and
:mod:`.multi` the one-process-per-GPU driver (shard + one allreduce).
"""
from . import hpl  # noqa: F401  (fails loudly if libhpl.so is missing)

__all__ = ["hpl"]
