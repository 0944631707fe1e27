"""B200-native Tahoe: batched decision-tree-ensemble prediction (EuroSys '21) on sm_100a.

The product is ``libtahoe.so`` (C ABI in include/tahoe.h); this package is its thin binding.
"""
from .tahoe import (AGG_AVERAGE, AGG_BINARY, AGG_CLASS_SUM, AGG_SUM, AGG_VOTE,  # noqa: F401
                    STRATEGY_AUTO, STRATEGY_DIRECT, STRATEGY_SLICED, Forest, TahoeError, load)
