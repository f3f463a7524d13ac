"""SNICIT sparse-DNN inference hot path on NVIDIA B200 (sm_100a).

The product is the C-ABI library ``lib/libsnicit.so`` (``include/snicit.h``); this package is its
thin Python binding (``api.SnicitNetwork``) plus row sharding / the category all-gather
(``parallel``).  No CPU fallback: the library must be built (``build.build()``).
"""
from ._lib import CSC as CSC_FORMAT, CSR as CSR_FORMAT  # noqa: F401
from ._lib import KERNEL_AUTO, KERNEL_CIRC, KERNEL_CIRC_SMEM, KERNEL_ELL, Options, SnicitError, default_options, load_library  # noqa: F401
from .api import SnicitNetwork, pack_rows, range_tables  # noqa: F401
from .parallel import (allgather_categories, allgather_categories_padded, assemble_categories,  # noqa: F401
                       shard_capacity, shard_rows)
