"""B200-native batched point-by-tree traversal (Goldfarb, Jo & Kulkarni, SC'13).

The hot path lives in libtt.so (hand-written CUDA for sm_100a behind the C ABI
of include/tt.h); this package is its thin Python binding (``tt``) plus the
multi-GPU driver (``parallel``).  Importing it loads libtt.so and fails loudly
if it has not been built -- there is no CPU fallback.
"""
from . import _lib
from ._lib import TTError

_lib.load()

from . import tt  # noqa: E402
from .tt import *  # noqa: E402,F401,F403
from . import nbody  # noqa: E402
from .nbody import tt_kick_drift, tt_kick_drift_permuted  # noqa: E402,F401

__all__ = ["tt", "nbody", "TTError", "tt_kick_drift", "tt_kick_drift_permuted"] + list(tt.__all__)
