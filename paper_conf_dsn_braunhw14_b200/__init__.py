"""B200-native (sm_100a) A-ABFT: checksum-protected GEMM with autonomous rounding-error bounds.

Braun, Halder, Wunderlich, DSN 2014.  The compute path is the C-ABI library libaabft.so
(include/aabft.h); this package is its thin torch binding (api), the row-sharded multi-GPU
driver (distributed) and the in-tree build (build).
"""
from ._abi import AabftError, COUNT_NAMES, STATUS_NAMES, launch_count, lib  # noqa: F401

__all__ = ["AabftError", "COUNT_NAMES", "STATUS_NAMES", "launch_count", "lib", "api",
           "distributed"]


def __getattr__(name):
    if name in ("api", "distributed"):
        import importlib
        return importlib.import_module(f".{name}", __name__)
    if name in ("ProtectedGemm", "protected_matmul", "gemm_plain"):
        from . import api
        return getattr(api, name)
    raise AttributeError(name)
