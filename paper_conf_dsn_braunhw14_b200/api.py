"""Thin torch-facing binding of the C ABI (include/aabft.h).

Torch provides device memory and the current CUDA stream; every step of the A-ABFT path
(encode, GEMM, bound, check, correct) runs in the sm_100a kernels of libaabft.so.  This
module only allocates buffers, builds the ABI structs and forwards pointers.

    plan = ProtectedGemm(M, N, K, dtype=torch.float64, bs=64, p=2)
    res = plan.run(A, B)             # A, B: CUDA tensors, row-major
    res.C, res.counts(), res.reports()

``protected_matmul(A, B, ...)`` is the one-shot convenience form (SURVEY §8(b) Python layer).
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass

import numpy as np
import torch

from . import _abi
from ._abi import Config, Encoded, Fault, Product, ok, lib

__all__ = ["ProtectedGemm", "protected_matmul", "gemm_plain", "make_faults", "make_faults_arrays",
           "counts_dict"]


def _dtype_code(dt: torch.dtype) -> int:
    if dt == torch.float64:
        return _abi.F64
    if dt == torch.float32:
        return _abi.F32
    raise TypeError("A-ABFT path supports torch.float64 and torch.float32")


def _pad_ld(n: int, dt: torch.dtype) -> int:
    q = 16 // torch.empty((), dtype=dt).element_size()
    return (n + q - 1) // q * q


def _stream_ptr(stream) -> int:
    s = torch.cuda.current_stream() if stream is None else stream
    return s.cuda_stream


def _ptr(t) -> int | None:
    return None if t is None else t.data_ptr()


def make_faults(faults, device) -> torch.Tensor | None:
    """List of dicts (row, col, site, k_step, xor_mask, add) -> device array of aabft_fault."""
    if not faults:
        return None
    arr = np.zeros(len(faults), dtype=_abi.FAULT_DTYPE)
    for n, f in enumerate(faults):
        arr[n]["row"] = f["row"]
        arr[n]["col"] = f["col"]
        arr[n]["site"] = f.get("site", 0)
        arr[n]["k_step"] = f.get("k_step", 0)
        arr[n]["xor_mask"] = np.uint64(f.get("xor_mask", 0))
        arr[n]["add"] = f.get("add", 0.0)
    return torch.from_numpy(arr.view(np.uint8).copy()).to(device)


def make_faults_arrays(row, col, site, k_step=0, xor_mask=0, add=0.0, device="cuda"):
    """Vectorised make_faults: equal-length arrays (or scalars) -> device aabft_fault array."""
    row = np.asarray(row, dtype=np.int64)
    arr = np.zeros(row.size, dtype=_abi.FAULT_DTYPE)
    arr["row"] = row
    arr["col"] = np.asarray(col, dtype=np.int64)
    arr["site"] = np.asarray(site, dtype=np.int32)
    arr["k_step"] = np.asarray(k_step, dtype=np.int64)
    arr["xor_mask"] = np.asarray(xor_mask, dtype=np.uint64)
    arr["add"] = np.asarray(add, dtype=np.float64)
    return torch.from_numpy(arr.view(np.uint8).copy()).to(device)


def counts_dict(counts: torch.Tensor) -> dict:
    """Decode an aabft_counts buffer (torch int64[9]) copied to the host."""
    c = counts.detach().cpu()
    d = {name: int(c[i]) for i, name in enumerate(_abi.COUNT_NAMES)}
    d["max_ratio"] = float(c[8:9].view(torch.float64)[0])
    return d


@dataclass
class Result:
    C: torch.Tensor
    Ccol: torch.Tensor
    Crow: torch.Tensor
    Acs: torch.Tensor
    Bcs: torch.Tensor
    topA_val: torch.Tensor
    topA_idx: torch.Tensor
    topB_val: torch.Tensor
    topB_idx: torch.Tensor
    report_buf: torch.Tensor
    counts_buf: torch.Tensor
    bs: int

    def counts(self) -> dict:
        return counts_dict(self.counts_buf)

    def reports(self) -> np.ndarray:
        """Structured numpy array (M/bs, N/bs) with the aabft_block_report fields."""
        raw = self.report_buf.detach().cpu().numpy()
        nI = self.C.shape[0] // self.bs
        return raw.view(_abi.REPORT_DTYPE).reshape(nI, -1)


class ProtectedGemm:
    """Pre-allocated buffers + ABI structs for repeated protected GEMMs of one shape."""

    def __init__(self, M: int, N: int, K: int, *, dtype=torch.float64, bs: int = 64, p: int = 2,
                 omega: float = 3.0, t: int = 0, fma_model: int = 1, device=None,
                 fused: bool = True, topp_in_gemm: bool = False, overlap: bool = False):
        lib()  # fail loudly before allocating anything
        self.device = torch.device("cuda" if device is None else device)
        self.dtype = dtype
        self.M, self.N, self.K, self.bs, self.p = M, N, K, bs, p
        # AABFT_FLAG_OVERLAP_ENCODE (include/aabft.h): the encode runs concurrently with the
        # GEMM's data tiles (FP64, 16 <= bs <= 64, p <= 4; ignored elsewhere).  Bit-identical
        # results; the workspace is zero-filled once below, as the flag's contract requires.
        # Opt-in: measured slower on B200 (the encode's FP64 adds stall the GEMM's DMMA pipe,
        # DESIGN.md 8.11).
        self.overlap = bool(overlap and dtype == torch.float64 and 16 <= bs <= 64 and p <= 4)
        self.cfg = Config(_dtype_code(dtype), bs, M, N, K, p, t, omega, fma_model,
                          _abi.FLAG_OVERLAP_ENCODE if self.overlap else 0)
        # AABFT_FLAG_TOPP_IN_GEMM (include/aabft.h): run() lets the GEMM select the top-p
        # (opt-in: measured slower than selecting in the encode pass)
        self.topp_in_gemm = bool(topp_in_gemm)
        self.cfg_defer = Config(_dtype_code(dtype), bs, M, N, K, p, t, omega, fma_model,
                                _abi.FLAG_TOPP_IN_GEMM)
        # AABFT_FLAG_CHECK_CORRECTS: run(correct=True) corrects inside the check kernel
        self.cfg_cc = Config(_dtype_code(dtype), bs, M, N, K, p, t, omega, fma_model,
                             self.cfg.flags | _abi.FLAG_CHECK_CORRECTS)
        self._topp_pending = False
        dev, dt = self.device, dtype
        nI, nJ = M // bs, N // bs
        self.ld_acs = _pad_ld(K, dt)
        self.ld_bcs = _pad_ld(nJ, dt)
        self.ldc = _pad_ld(N, dt)
        self.ld_ccol = _pad_ld(N, dt)
        self.ld_crow = _pad_ld(nJ, dt)
        # zeroed once: the 16-byte pitch padding is then defined for the FP32 GEMM's 16-byte
        # cp.async row loads (compute-sanitizer initcheck clean; the padding never reaches C)
        self._Acs = torch.zeros(nI, self.ld_acs, dtype=dt, device=dev)
        self._Bcs = torch.zeros(K, self.ld_bcs, dtype=dt, device=dev)
        self._C = torch.empty(M, self.ldc, dtype=dt, device=dev)
        self._Ccol = torch.empty(nI, self.ld_ccol, dtype=dt, device=dev)
        self._Crow = torch.empty(M, self.ld_crow, dtype=dt, device=dev)
        self.topA_val = torch.empty(M + nI, p, dtype=torch.float64, device=dev)
        self.topA_idx = torch.empty(M + nI, p, dtype=torch.int32, device=dev)
        self.topB_val = torch.empty(N + nJ, p, dtype=torch.float64, device=dev)
        self.topB_idx = torch.empty(N + nJ, p, dtype=torch.int32, device=dev)
        self.reports = torch.empty(nI * nJ * 20, dtype=torch.uint8, device=dev)
        self.counts = torch.zeros(9, dtype=torch.int64, device=dev)
        wsb = lib().aabft_workspace_bytes(C.byref(self.cfg))
        if wsb == 0:
            ok(1, "aabft_workspace_bytes")
        self.ws_bytes = int(wsb)
        self.ws = torch.zeros(self.ws_bytes, dtype=torch.uint8, device=dev)
        self.enc = Encoded(self._Acs.data_ptr(), self.ld_acs, self._Bcs.data_ptr(), self.ld_bcs,
                           self.topA_val.data_ptr(), self.topA_idx.data_ptr(),
                           self.topB_val.data_ptr(), self.topB_idx.data_ptr())
        # checksums-only view (no top-p tables): the comparators' encoding (NEXT-3)
        self.enc_cs = Encoded(self._Acs.data_ptr(), self.ld_acs, self._Bcs.data_ptr(),
                              self.ld_bcs, None, None, None, None)
        self._sea = None
        # fused check (FP64 bs <= 64, FP32 bs <= 128): the GEMM epilogue writes the reference sums
        self.fused = bool(fused and ((dtype == torch.float64 and bs <= 64) or
                                     (dtype == torch.float32 and bs <= 128)))
        self.Rcol = torch.empty(nI, N, dtype=torch.float64, device=dev) if self.fused else None
        self.Rrow = torch.empty(M, nJ, dtype=torch.float64, device=dev) if self.fused else None
        self.prod = Product(self._C.data_ptr(), self.ldc, self._Ccol.data_ptr(), self.ld_ccol,
                            self._Crow.data_ptr(), self.ld_crow, _ptr(self.Rcol), _ptr(self.Rrow))

    # views without the pitch padding
    @property
    def C(self):
        return self._C[:, : self.N]

    @property
    def Ccol(self):
        return self._Ccol[:, : self.N]

    @property
    def Crow(self):
        return self._Crow[:, : self.N // self.bs]

    @property
    def Acs(self):
        return self._Acs[:, : self.K]

    @property
    def Bcs(self):
        return self._Bcs[:, : self.N // self.bs]

    def _check_operand(self, X, rows, cols, name):
        if not X.is_cuda or X.dtype != self.dtype or tuple(X.shape) != (rows, cols):
            raise ValueError(f"{name} must be a CUDA {self.dtype} tensor of shape {(rows, cols)}")
        if X.stride(1) != 1:
            raise ValueError(f"{name} must be row-major (stride(1) == 1)")

    # --- the four steps (each one C-ABI call)
    def encode(self, A, B, stream=None, topp: bool = True, defer: bool = False):
        """Step 1; topp=False encodes the checksums only (fixed-eps / SEA comparators);
        defer=True leaves the top-p selection to the following gemm() where the library
        supports it (AABFT_FLAG_TOPP_IN_GEMM; the tables are complete after gemm())."""
        L = lib()
        s = _stream_ptr(stream)
        self._topp_pending = bool(defer and topp)
        cfg = self.cfg_defer if self._topp_pending else self.cfg
        ok(L.aabft_encode(C.byref(cfg), _ptr(A), A.stride(0) if A is not None else 0,
                          _ptr(B), B.stride(0) if B is not None else 0,
                          C.byref(self.enc if topp else self.enc_cs),
                          self.ws.data_ptr(), self.ws_bytes, s), "aabft_encode")

    def gemm(self, A, B, faults: torch.Tensor | None = None, nfaults: int = 0, stream=None):
        cfg = self.cfg_defer if self._topp_pending else self.cfg
        self._topp_pending = False
        ok(lib().aabft_gemm(C.byref(cfg), A.data_ptr(), A.stride(0), B.data_ptr(),
                            B.stride(0), C.byref(self.enc), C.byref(self.prod), _ptr(faults),
                            nfaults, self.ws.data_ptr(), self.ws_bytes, _stream_ptr(stream)),
           "aabft_gemm")

    def check(self, stream=None, correct: bool = False):
        """Step 3; correct=True also corrects the located single errors in the same kernel
        (AABFT_FLAG_CHECK_CORRECTS), which makes correct() unnecessary."""
        cfg = self.cfg_cc if correct else self.cfg
        ok(lib().aabft_check(C.byref(cfg), C.byref(self.enc), C.byref(self.prod),
                             self.reports.data_ptr(), self.counts.data_ptr(), self.ws.data_ptr(),
                             self.ws_bytes, _stream_ptr(stream)), "aabft_check")

    def correct(self, stream=None):
        ok(lib().aabft_correct(C.byref(self.cfg), C.byref(self.enc), C.byref(self.prod),
                               self.reports.data_ptr(), self.counts.data_ptr(),
                               _stream_ptr(stream)), "aabft_correct")

    def bound(self, stream=None):
        nI, nJ = self.M // self.bs, self.N // self.bs
        eps_col = torch.empty(nI, self.N, dtype=torch.float64, device=self.device)
        sig_col = torch.empty_like(eps_col)
        eps_row = torch.empty(self.M, nJ, dtype=torch.float64, device=self.device)
        sig_row = torch.empty_like(eps_row)
        ok(lib().aabft_bound(C.byref(self.cfg), C.byref(self.enc), eps_col.data_ptr(),
                             sig_col.data_ptr(), eps_row.data_ptr(), sig_row.data_ptr(),
                             _stream_ptr(stream)), "aabft_bound")
        return dict(eps_col=eps_col, sig_col=sig_col, eps_row=eps_row, sig_row=sig_row)

    def bound_elements(self, rows, cols, stream=None):
        """sigma, eps of arbitrary C_fc elements; rows/cols: int64 CUDA tensors."""
        rows = rows.to(device=self.device, dtype=torch.int64).contiguous()
        cols = cols.to(device=self.device, dtype=torch.int64).contiguous()
        n = rows.numel()
        sig = torch.empty(n, dtype=torch.float64, device=self.device)
        eps = torch.empty(n, dtype=torch.float64, device=self.device)
        ok(lib().aabft_bound_elements(C.byref(self.cfg), C.byref(self.enc), rows.data_ptr(),
                                      cols.data_ptr(), n, sig.data_ptr(), eps.data_ptr(),
                                      _stream_ptr(stream)), "aabft_bound_elements")
        return sig, eps

    def checksum_errors(self, A, B, stream=None):
        """carried - exact (double-double) for every carried checksum (NEXT-1, Tables II/III)."""
        nI, nJ = self.M // self.bs, self.N // self.bs
        err_col = torch.empty(nI, self.N, dtype=torch.float64, device=self.device)
        err_row = torch.empty(self.M, nJ, dtype=torch.float64, device=self.device)
        ok(lib().aabft_checksum_errors(C.byref(self.cfg), A.data_ptr(), A.stride(0), B.data_ptr(),
                                       B.stride(0), C.byref(self.enc), C.byref(self.prod),
                                       err_col.data_ptr(), err_row.data_ptr(), _stream_ptr(stream)),
           "aabft_checksum_errors")
        return err_col, err_row

    # --- NEXT-3 comparators (reporting only)
    def sea_bound(self, A, B, *, corner: bool = False, stream=None) -> dict:
        """SEA-ABFT eps of every carried checksum (§III); needs encode() first."""
        nI, nJ = self.M // self.bs, self.N // self.bs
        if self._sea is None:
            self._sea = dict(
                eps_col=torch.empty(nI, self.N, dtype=torch.float64, device=self.device),
                eps_row=torch.empty(self.M, nJ, dtype=torch.float64, device=self.device),
                eps_corner=torch.empty(nI, nJ, dtype=torch.float64, device=self.device))
        d = self._sea
        ok(lib().aabft_sea_bound(C.byref(self.cfg), A.data_ptr(), A.stride(0), B.data_ptr(),
                                 B.stride(0), C.byref(self.enc_cs), d["eps_col"].data_ptr(),
                                 d["eps_row"].data_ptr(),
                                 d["eps_corner"].data_ptr() if corner else None,
                                 self.ws.data_ptr(), self.ws_bytes, _stream_ptr(stream)),
           "aabft_sea_bound")
        return d

    def check_ext(self, *, eps_col=None, eps_row=None, eps_fixed: float = 0.0, stream=None):
        ok(lib().aabft_check_ext(C.byref(self.cfg), C.byref(self.prod), _ptr(eps_col),
                                 _ptr(eps_row), float(eps_fixed), self.reports.data_ptr(),
                                 self.counts.data_ptr(), self.ws.data_ptr(), self.ws_bytes,
                                 _stream_ptr(stream)), "aabft_check_ext")

    def correct_ext(self, *, eps_row=None, eps_fixed: float = 0.0, stream=None):
        ok(lib().aabft_correct_ext(C.byref(self.cfg), C.byref(self.prod), _ptr(eps_row),
                                   float(eps_fixed), self.reports.data_ptr(),
                                   self.counts.data_ptr(), _stream_ptr(stream)),
           "aabft_correct_ext")

    def run_ext(self, A, B, *, mode: str = "sea", eps_fixed: float = 0.0, faults=None,
                correct: bool = True, stream=None) -> Result:
        """Comparator paths of Table I: checksums-only encode -> GEMM -> check /
        correct against the SEA-ABFT bound (mode "sea") or one fixed eps (mode "fixed")."""
        if mode not in ("sea", "fixed"):
            raise ValueError(mode)
        self._check_operand(A, self.M, self.K, "A")
        self._check_operand(B, self.K, self.N, "B")
        fbuf = faults if isinstance(faults, torch.Tensor) else make_faults(faults, self.device)
        nf = 0 if fbuf is None else fbuf.numel() // 48
        self.encode(A, B, stream, topp=False)
        ok(lib().aabft_gemm(C.byref(self.cfg), A.data_ptr(), A.stride(0), B.data_ptr(),
                            B.stride(0), C.byref(self.enc_cs), C.byref(self.prod), _ptr(fbuf),
                            nf, self.ws.data_ptr(), self.ws_bytes, _stream_ptr(stream)),
           "aabft_gemm")
        ec = er = None
        if mode == "sea":
            d = self.sea_bound(A, B, stream=stream)
            ec, er = d["eps_col"], d["eps_row"]
        self.check_ext(eps_col=ec, eps_row=er, eps_fixed=eps_fixed, stream=stream)
        if correct:
            self.correct_ext(eps_row=er, eps_fixed=eps_fixed, stream=stream)
        return self.result()

    def run(self, A, B, *, faults=None, correct: bool = True, stream=None) -> Result:
        """encode -> gemm -> check + correct, all enqueued on one stream; the
        correction of located single errors runs inside the check kernel."""
        self._check_operand(A, self.M, self.K, "A")
        self._check_operand(B, self.K, self.N, "B")
        fbuf = faults if isinstance(faults, torch.Tensor) else make_faults(faults, self.device)
        nf = 0 if fbuf is None else fbuf.numel() // 48
        self.encode(A, B, stream, defer=self.topp_in_gemm)
        self.gemm(A, B, fbuf, nf, stream)
        self.check(stream, correct=correct)  # correction fused into the check kernel
        return self.result()

    def capture(self, A, B, *, correct: bool = True):
        """Record encode -> gemm -> check -> correct for these (fixed) A, B buffers as one CUDA
        graph; ``graph.replay()`` re-runs the whole protected product (new contents of A and B
        are picked up).  For launch-latency-bound sizes (BASELINE configs[0]: 128^3 is ~10 us
        of GPU work against ~8 launches).  The first eager run sets the kernels' one-time
        attributes outside the capture."""
        side = torch.cuda.Stream(self.device)
        side.wait_stream(torch.cuda.current_stream(self.device))
        with torch.cuda.stream(side):
            self.run(A, B, correct=correct)
        torch.cuda.current_stream(self.device).wait_stream(side)
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            self.run(A, B, correct=correct)
        return graph

    def result(self) -> Result:
        return Result(self.C, self.Ccol, self.Crow, self.Acs, self.Bcs, self.topA_val,
                      self.topA_idx, self.topB_val, self.topB_idx, self.reports, self.counts,
                      self.bs)


def protected_matmul(A, B, *, bs: int = 64, p: int = 2, omega: float = 3.0, t: int = 0,
                     fma_model: int = 1, correct: bool = True, faults=None) -> Result:
    """One-shot A-ABFT protected C = A @ B on the current CUDA stream."""
    M, K = A.shape
    N = B.shape[1]
    plan = ProtectedGemm(M, N, K, dtype=A.dtype, bs=bs, p=p, omega=omega, t=t,
                         fma_model=fma_model, device=A.device)
    return plan.run(A, B, faults=faults, correct=correct)


_plain_ws = {}


def gemm_plain(A, B, out=None, stream=None):
    """Unprotected C = A @ B with the same kernel family and scheduler (overhead denominator)."""
    M, K = A.shape
    N = B.shape[1]
    dt = A.dtype
    if M % 8 or N % 8:
        raise ValueError("gemm_plain: M and N must be multiples of 8")
    if out is None:
        out = torch.empty(M, _pad_ld(N, dt), dtype=dt, device=A.device)
    cfg = Config(_dtype_code(dt), 8, M, N, K, 1, 0, 3.0, 1, 0)  # bs=8: validation only
    wsb = int(lib().aabft_gemm_plain_workspace_bytes(C.byref(cfg)))
    key = (A.device, wsb)
    if key not in _plain_ws:
        _plain_ws.clear()
        _plain_ws[key] = torch.empty(wsb, dtype=torch.uint8, device=A.device)
    ws = _plain_ws[key]
    ok(lib().aabft_gemm_plain(C.byref(cfg), A.data_ptr(), A.stride(0), B.data_ptr(), B.stride(0),
                              out.data_ptr(), out.stride(0), ws.data_ptr(), wsb,
                              _stream_ptr(stream)), "aabft_gemm_plain")
    return out[:, :N]
