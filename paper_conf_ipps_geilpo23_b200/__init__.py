"""B200-native breadth-first maximum clique enumeration (Geil, Porumbescu &
Owens, IPDPS 2023) -- hand-written sm_100a CUDA behind a C ABI
(include/mce.h), this package is its thin Python binding.

Importing the package does not load the CUDA library; the first call does,
and raises if libmce_b200.so is missing (there is no CPU fallback).
"""

from .api import Graph, Result, empty_cache, make_options, version  # noqa: F401
from ._lib import MCEError, build  # noqa: F401
from .distributed import enumerate_distributed, find_one_distributed  # noqa: F401
