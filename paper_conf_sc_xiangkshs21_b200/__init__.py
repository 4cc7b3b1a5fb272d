"""cuTS hot path on B200: trie-based subgraph-isomorphism search (Xiang et al., SC '21).

The package is a thin binding over ``libcuts.so`` (CUDA, sm_100a; C ABI in
``include/cuts.h``).  Importing it loads the shared library and fails loudly if
it is missing — there is no CPU fallback.
"""
from . import _lib
from ._lib import load as _load_lib

_load_lib()

from .api import Cuts, CutsError, default_arena_bytes  # noqa: E402

__all__ = ["Cuts", "CutsError", "default_arena_bytes"]
