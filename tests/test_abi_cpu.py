"""C-ABI library checks that need no GPU: it loads, exports every symbol include/aabft.h
declares, and rejects invalid arguments before touching a device (no compute calls)."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "aabft.h")).read()
    decl = r"^\s*(?:const\s+)?[a-z_0-9]+\s*\*?\s*(aabft_[a-z_]+)\s*\("
    return sorted(set(re.findall(decl, src, re.MULTILINE)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_dsn_braunhw14_b200 import build as b
    b.build()
    from paper_conf_dsn_braunhw14_b200 import _abi
    return _abi.lib()


def test_header_declares_the_path():
    names = _declared()
    for n in ("aabft_encode", "aabft_gemm", "aabft_check", "aabft_correct", "aabft_bound",
              "aabft_gemm_plain", "aabft_workspace_bytes"):
        assert n in names


def test_every_declared_symbol_is_exported(L):
    for n in _declared():
        assert hasattr(L, n), n
    from paper_conf_dsn_braunhw14_b200 import _abi
    assert set(_abi.EXPORTED) == set(_declared())


def test_struct_layout_matches_header(tmp_path):
    """ctypes mirror == the C compiler's layout of include/aabft.h (sizes and offsets)."""
    import subprocess
    from paper_conf_dsn_braunhw14_b200 import _abi
    checks = {"aabft_config": (_abi.Config, ["dtype", "bs", "M", "N", "K", "p", "t", "omega",
                                             "fma_model"]),
              "aabft_encoded": (_abi.Encoded, ["Acs", "ld_acs", "Bcs", "ld_bcs", "topA_val",
                                               "topA_idx", "topB_val", "topB_idx"]),
              "aabft_product": (_abi.Product, ["C", "ldc", "Ccol", "ld_ccol", "Crow", "ld_crow",
                                               "Rcol", "Rrow"]),
              "aabft_block_report": (_abi.BlockReport, ["status", "worst_class", "n_bad_rows",
                                                        "n_bad_cols", "row", "col", "max_ratio"]),
              "aabft_counts": (_abi.Counts, ["n", "max_ratio"]),
              "aabft_fault": (_abi.Fault, ["row", "col", "site", "k_step", "xor_mask", "add"])}
    lines = ['#include <stdio.h>', '#include <stddef.h>', '#include "aabft.h"', "int main(void){"]
    for st, (_, fields) in checks.items():
        lines.append(f'printf("{st} %zu\\n", sizeof({st}));')
        for f in fields:
            lines.append(f'printf("{st}.{f} %zu\\n", offsetof({st}, {f}));')
    lines.append("return 0;}")
    src = tmp_path / "layout.c"
    src.write_text("\n".join(lines))
    exe = tmp_path / "layout"
    subprocess.check_call(["gcc", "-I", os.path.join(ROOT, "include"), str(src), "-o", str(exe)])
    got = dict(l.split() for l in subprocess.check_output([str(exe)]).decode().splitlines())
    for st, (cls, fields) in checks.items():
        assert int(got[st]) == C.sizeof(cls), st
        for f in fields:
            assert int(got[f"{st}.{f}"]) == getattr(cls, f).offset, (st, f)
    assert _abi.REPORT_DTYPE.itemsize == int(got["aabft_block_report"])
    assert _abi.FAULT_DTYPE.itemsize == int(got["aabft_fault"])


def _cfg(**kw):
    from paper_conf_dsn_braunhw14_b200 import _abi
    d = dict(dtype=0, bs=64, M=256, N=256, K=256, p=2, t=0, omega=3.0, fma_model=1)
    d.update(kw)
    return _abi.Config(d["dtype"], d["bs"], d["M"], d["N"], d["K"], d["p"], d["t"], d["omega"],
                       d["fma_model"], 0)


@pytest.mark.parametrize("bad", [dict(M=0), dict(K=0), dict(bs=48), dict(bs=4), dict(bs=512),
                                 dict(M=100), dict(N=72), dict(p=0), dict(p=9),
                                 dict(K=1, p=2), dict(omega=0.0), dict(omega=float("nan")),
                                 dict(dtype=7), dict(fma_model=2), dict(t=-1)])
def test_invalid_config_rejected(L, bad):
    cfg = _cfg(**bad)
    assert L.aabft_workspace_bytes(C.byref(cfg)) == 0
    from paper_conf_dsn_braunhw14_b200 import _abi
    enc = _abi.Encoded()
    st = L.aabft_encode(C.byref(cfg), 16, 256, 16, 256, C.byref(enc), 16, 1 << 20, None)
    assert st == 1  # AABFT_EINVAL
    assert len(L.aabft_last_error()) > 0


def test_workspace_and_null_checks(L):
    from paper_conf_dsn_braunhw14_b200 import _abi
    cfg = _cfg()
    assert L.aabft_workspace_bytes(C.byref(cfg)) > 0
    assert L.aabft_host_arena_bytes(C.byref(cfg)) > 3 * 256 * 256 * 8
    enc = _abi.Encoded()
    # both operands NULL
    assert L.aabft_encode(C.byref(cfg), None, 256, None, 256, C.byref(enc), 16, 1 << 20, None) == 1
    # lda < K
    enc = _abi.Encoded(16, 256, 16, 4, 16, 16, 16, 16)
    assert L.aabft_encode(C.byref(cfg), 16, 100, None, 0, C.byref(enc), 16, 1 << 20, None) == 1
    # workspace too small
    assert L.aabft_encode(C.byref(cfg), 16, 256, None, 0, C.byref(enc), 16, 8, None) == 4
    # misaligned operand for the TMA GEMM
    prod = _abi.Product(16, 256, 16, 256, 16, 4, None, None)
    st = L.aabft_gemm(C.byref(cfg), 8, 256, 16, 256, C.byref(enc), C.byref(prod), None, 0, 16,
                      1 << 40, None)
    assert st == 1 and b"aligned" in L.aabft_last_error()
    assert L.aabft_status_str(4).startswith(b"AABFT_EWORKSPACE")
    assert L.aabft_version().startswith(b"aabft-b200")


def test_comparator_entry_points_validate(L):
    """NEXT-3 comparators: argument checks run before any device access."""
    from paper_conf_dsn_braunhw14_b200 import _abi
    cfg = _cfg()
    enc = _abi.Encoded(16, 256, 16, 4, None, None, None, None)
    # only one of the top-p pair: invalid
    half = _abi.Encoded(16, 256, 16, 4, 16, None, None, None)
    assert L.aabft_encode(C.byref(cfg), 16, 256, None, 0, C.byref(half), 16, 1 << 20, None) == 1
    # SEA bound: no output / missing operand / workspace too small
    assert L.aabft_sea_bound(C.byref(cfg), 16, 256, 16, 256, C.byref(enc), None, None, None, 16,
                             1 << 20, None) == 1
    assert L.aabft_sea_bound(C.byref(cfg), None, 256, 16, 256, C.byref(enc), 16, None, None, 16,
                             1 << 20, None) == 1
    assert L.aabft_sea_bound(C.byref(cfg), 16, 256, 16, 256, C.byref(enc), 16, None, None, 16,
                             8, None) == 4
    # external-eps check: negative / NaN eps_fixed, missing buffers
    prod = _abi.Product(16, 256, 16, 256, 16, 4, None, None)
    for bad in (-1.0, float("nan")):
        assert L.aabft_check_ext(C.byref(cfg), C.byref(prod), None, None, bad, 16, 16, None, 0,
                                 None) == 1
    assert L.aabft_check_ext(C.byref(cfg), C.byref(prod), None, None, 1.0, None, 16, None, 0,
                             None) == 1
    assert L.aabft_correct_ext(C.byref(cfg), None, None, 1.0, 16, 16, None) == 1


def test_product_path_has_no_oracle_import():
    """The product package never imports or loads anything under oracle/ (no CPU fallback)."""
    pkg = os.path.join(ROOT, "paper_conf_dsn_braunhw14_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                for pat in ("import oracle", "from oracle", "libaabft_oracle", "aabft_oracle"):
                    assert pat not in src, (f, pat)
