"""pc — GPU-initiated MPI-Partitioned-style communication for B200.

From-scratch, B200-native rebuild of the data-parallel hot path of Temuçin et
al., SC'24 (intra-kernel GPU-initiated partitioned p2p, partitioned allreduce,
Jacobi with intra-kernel partitioned halos).  The product is the C-ABI library
``libpc.so`` (include/pc.h, include/pc_device.cuh); this package is its thin
ctypes binding.  There is no CPU fallback: a missing library raises.
"""
from .runtime import *  # noqa: F401,F403
from .runtime import Comm, LocalGroup, PcError, Prequest, Request, local_comms, run_ranks  # noqa: F401
from . import _lib  # noqa: F401

__version__ = "0.1.0"
