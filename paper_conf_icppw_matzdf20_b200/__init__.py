"""B200-native partitioned-kernel runtime (hot path of Matz/Doerfert/Fröning, ICPPW 2020).

The product is the C-ABI library ``libpk.so`` (include/pk_api.h); ``abi`` is its
thin ctypes binding with the same function names and ``kernels`` holds the
launch geometry of the builtin sm_100a kernels.  There is no CPU fallback.
"""
from . import abi  # noqa: F401
from .abi import *  # noqa: F401,F403

__all__ = [n for n in dir(abi) if n.startswith("pk_") or n.startswith("PK_")]
