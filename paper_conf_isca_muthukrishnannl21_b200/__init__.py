"""PROACT hot path on B200 (sm_100a): C-ABI library libproact + thin Python binding.

Paper: Muthukrishnan, Nellans, Lustig, Fessler, Wenisch, "Efficient Multi-GPU
Shared Memory via Automatic Optimization of Fine-Grained Transfers", ISCA 2021.
See DESIGN.md for the path, its boundary (include/*.h) and the readings taken.
"""
import os as _os

# The agent kernel runs on its own high-priority stream; with the default 8 hardware queues its
# launches can wait behind the producer stream (false dependencies).  Effective only if this
# package is imported before anything creates a CUDA context (bench.py sets it before torch).
_os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

from . import _lib  # noqa: E402
from ._lib import (MECH_BULK, MECH_ELIDE, MECH_FUSED, MECH_INLINE, MECH_LOCAL, MECH_NAMES,
                   REGION_SPARSE, ProactError)
from . import runtime
from . import workloads
from .loopback import run_ranks

__all__ = ["runtime", "workloads", "run_ranks", "ProactError", "MECH_FUSED", "MECH_INLINE",
           "MECH_BULK", "MECH_LOCAL", "MECH_ELIDE", "MECH_NAMES", "REGION_SPARSE", "load"]


def load():
    """Load libproact.so; raises ImportError if it is missing (no CPU fallback)."""
    return _lib.load()
