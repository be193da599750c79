"""ctypes mirror of include/aabft.h (argument marshalling only; no method arithmetic here).

The CUDA library is REQUIRED: if ``libaabft.so`` is missing or fails to load, every entry
point raises -- there is no CPU fallback anywhere on the product path.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
# AABFT_LIB selects an alternative build of the same library (tuning experiments only)
LIB_PATH = os.environ.get("AABFT_LIB", os.path.join(HERE, "libaabft.so"))

F64, F32 = 0, 1
BLK_CLEAN, BLK_CORRECTED, BLK_CHECKSUM_ONLY, BLK_UNCORRECTABLE, BLK_SINGLE = 0, 1, 2, 3, 4
STATUS_NAMES = {0: "CLEAN", 1: "CORRECTED", 2: "CHECKSUM_ONLY", 3: "UNCORRECTABLE", 4: "SINGLE"}
FLAG_TOPP_IN_GEMM = 1  # include/aabft.h AABFT_FLAG_TOPP_IN_GEMM
FLAG_GEMM_HALF_GRID = 2  # AABFT_FLAG_GEMM_HALF_GRID
FLAG_OVERLAP_ENCODE = 4  # AABFT_FLAG_OVERLAP_ENCODE
FLAG_CHECK_CORRECTS = 8  # AABFT_FLAG_CHECK_CORRECTS
COUNT_NAMES = ("blocks", "clean", "corrected", "checksum_only", "uncorrectable",
               "checks_rounding", "checks_tolerable", "checks_critical")
EXPORTED = ("aabft_workspace_bytes", "aabft_encode", "aabft_bound", "aabft_bound_elements",
            "aabft_gemm",
            "aabft_gemm_plain", "aabft_check", "aabft_correct", "aabft_host_arena_bytes",
            "aabft_protected_gemm_host", "aabft_status_str", "aabft_last_error",
            "aabft_version", "aabft_launch_count", "aabft_checksum_errors", "aabft_sea_bound",
            "aabft_check_ext", "aabft_correct_ext", "aabft_gemm_plain_workspace_bytes")


class Config(C.Structure):
    _fields_ = [("dtype", C.c_int32), ("bs", C.c_int32), ("M", C.c_int64), ("N", C.c_int64),
                ("K", C.c_int64), ("p", C.c_int32), ("t", C.c_int32), ("omega", C.c_double),
                ("fma_model", C.c_int32), ("flags", C.c_int32)]


class Encoded(C.Structure):
    _fields_ = [("Acs", C.c_void_p), ("ld_acs", C.c_int64), ("Bcs", C.c_void_p),
                ("ld_bcs", C.c_int64), ("topA_val", C.c_void_p), ("topA_idx", C.c_void_p),
                ("topB_val", C.c_void_p), ("topB_idx", C.c_void_p)]


class Product(C.Structure):
    _fields_ = [("C", C.c_void_p), ("ldc", C.c_int64), ("Ccol", C.c_void_p),
                ("ld_ccol", C.c_int64), ("Crow", C.c_void_p), ("ld_crow", C.c_int64),
                ("Rcol", C.c_void_p), ("Rrow", C.c_void_p)]


class BlockReport(C.Structure):
    _fields_ = [("status", C.c_uint8), ("worst_class", C.c_uint8), ("n_bad_rows", C.c_uint16),
                ("n_bad_cols", C.c_uint16), ("reserved", C.c_uint16), ("row", C.c_int32),
                ("col", C.c_int32), ("max_ratio", C.c_float)]


class Counts(C.Structure):
    _fields_ = [("n", C.c_int64 * 8), ("max_ratio", C.c_double)]


class Fault(C.Structure):
    _fields_ = [("row", C.c_int64), ("col", C.c_int64), ("site", C.c_int32),
                ("reserved", C.c_int32), ("k_step", C.c_int64), ("xor_mask", C.c_uint64),
                ("add", C.c_double)]


REPORT_DTYPE = np.dtype({"names": ["status", "worst_class", "n_bad_rows", "n_bad_cols", "reserved",
                                   "row", "col", "max_ratio"],
                         "formats": [np.uint8, np.uint8, np.uint16, np.uint16, np.uint16, np.int32,
                                     np.int32, np.float32],
                         "offsets": [0, 1, 2, 4, 6, 8, 12, 16], "itemsize": 20})
FAULT_DTYPE = np.dtype({"names": ["row", "col", "site", "reserved", "k_step", "xor_mask", "add"],
                        "formats": [np.int64, np.int64, np.int32, np.int32, np.int64, np.uint64,
                                    np.float64],
                        "offsets": [0, 8, 16, 20, 24, 32, 40], "itemsize": 48})
assert C.sizeof(BlockReport) == 20 and C.sizeof(Fault) == 48 and C.sizeof(Counts) == 72

_lib = None


class AabftError(RuntimeError):
    pass


def lib():
    """Load libaabft.so (in-tree).  Raises if it is missing: no fallback exists."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise AabftError(f"{LIB_PATH} not built; run __graft_entry__.build() "
                             "(python -m paper_conf_dsn_braunhw14_b200.build)")
        L = C.CDLL(LIB_PATH)
        vp, i64, i32, sz = C.c_void_p, C.c_int64, C.c_int32, C.c_size_t
        pc = C.POINTER(Config)
        L.aabft_workspace_bytes.argtypes = [pc]
        L.aabft_workspace_bytes.restype = sz
        L.aabft_gemm_plain_workspace_bytes.argtypes = [pc]
        L.aabft_gemm_plain_workspace_bytes.restype = sz
        L.aabft_host_arena_bytes.argtypes = [pc]
        L.aabft_host_arena_bytes.restype = sz
        L.aabft_encode.argtypes = [pc, vp, i64, vp, i64, C.POINTER(Encoded), vp, sz, vp]
        L.aabft_bound.argtypes = [pc, C.POINTER(Encoded), vp, vp, vp, vp, vp]
        L.aabft_bound_elements.argtypes = [pc, C.POINTER(Encoded), vp, vp, i64, vp, vp, vp]
        L.aabft_checksum_errors.argtypes = [pc, vp, i64, vp, i64, C.POINTER(Encoded),
                                            C.POINTER(Product), vp, vp, vp]
        L.aabft_gemm.argtypes = [pc, vp, i64, vp, i64, C.POINTER(Encoded), C.POINTER(Product), vp,
                                 i32, vp, sz, vp]
        L.aabft_gemm_plain.argtypes = [pc, vp, i64, vp, i64, vp, i64, vp, sz, vp]
        L.aabft_check.argtypes = [pc, C.POINTER(Encoded), C.POINTER(Product), vp, vp, vp, sz, vp]
        L.aabft_correct.argtypes = [pc, C.POINTER(Encoded), C.POINTER(Product), vp, vp, vp]
        L.aabft_protected_gemm_host.argtypes = [pc, vp, vp, vp, vp, vp, sz, vp]
        L.aabft_sea_bound.argtypes = [pc, vp, i64, vp, i64, C.POINTER(Encoded), vp, vp, vp, vp,
                                      sz, vp]
        L.aabft_check_ext.argtypes = [pc, C.POINTER(Product), vp, vp, C.c_double, vp, vp, vp, sz,
                                      vp]
        L.aabft_correct_ext.argtypes = [pc, C.POINTER(Product), vp, C.c_double, vp, vp, vp]
        L.aabft_status_str.argtypes = [C.c_int]
        L.aabft_status_str.restype = C.c_char_p
        L.aabft_last_error.restype = C.c_char_p
        L.aabft_version.restype = C.c_char_p
        L.aabft_launch_count.restype = i64
        for name in ("aabft_encode", "aabft_bound", "aabft_bound_elements", "aabft_checksum_errors",
                     "aabft_gemm", "aabft_gemm_plain",
                     "aabft_check", "aabft_correct", "aabft_protected_gemm_host",
                     "aabft_sea_bound", "aabft_check_ext", "aabft_correct_ext"):
            getattr(L, name).restype = C.c_int
        _lib = L
    return _lib


def ok(status: int, what: str) -> None:
    if status != 0:
        L = lib()
        raise AabftError(f"{what}: {L.aabft_status_str(status).decode()} -- "
                         f"{L.aabft_last_error().decode()}")


def launch_count() -> int:
    return int(lib().aabft_launch_count())
