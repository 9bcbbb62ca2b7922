"""paper_conf_hpdc_raschg18_b200 — B200-native ATF search-space generation.

The hot path of ATF (Rasch, Haidl & Gorlatch, HPCC 2017): generating the search
space of interdependent tuning parameters (§II Step 1, §V, §VI-A) as
hand-written sm_100a kernels behind a C ABI (include/atfgen.h).  This package is
the thin Python binding (``_lib``: the C functions; ``space.Space``: marshalling)
and the multi-GPU glue (``shard``: counts all-gather over torch.distributed).  Importing it requires the built
``libatfgen.so``; there is no CPU fallback.
"""
from . import _lib  # noqa: F401  (raises ImportError if the CUDA library is missing)
from ._lib import AtfError  # noqa: F401
from .space import Space  # noqa: F401

__all__ = ["Space", "AtfError"]
