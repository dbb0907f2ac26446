"""C-ABI contract checks that need no GPU: the library loads, exports every symbol
include/fmha.h declares, and host-side validation returns the documented status codes
before anything would be launched."""

import ctypes
import os
import re
import subprocess

import pytest

from paper_conf_asplos_hagedornfccgg23_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "fmha.h")


@pytest.fixture(scope="module")
def lib():
    if not os.path.exists(_lib.LIB_PATH):
        subprocess.run(["make", "-C", os.path.join(ROOT, "paper_conf_asplos_hagedornfccgg23_b200")], check=True)
    return _lib.load()


def header_functions():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"^\s*FMHA_API\s+(?:const\s+)?[a-z_0-9]+\s*\*?\s*([a-z_0-9]+)\s*\(", txt, flags=re.M)))


def test_header_declares_expected_symbols():
    assert sorted(_lib.EXPORTED_SYMBOLS) == header_functions()


def test_every_declared_symbol_is_exported(lib):
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIB_PATH], capture_output=True, text=True).stdout
    exported = {ln.split()[-1] for ln in out.splitlines() if ln.strip()}
    for name in header_functions():
        assert name in exported, name
        assert getattr(lib, name) is not None


def test_status_strings(lib):
    for code, name in _lib.STATUS_NAMES.items():
        assert lib.fmha_status_string(code).decode().startswith(name)
    assert lib.fmha_version().decode().startswith("b200fmha")


def call_fmha(lib, q=16, k=16, v=16, o=16, mask=None, b=1, h=1, sq=8, skv=8, d=64, scale=0.125):
    m = ctypes.byref(mask) if mask is not None else None
    return lib.fmha_fwd(q, k, v, o, m, b, h, sq, skv, d, scale, None)


def test_validation_codes(lib):
    assert call_fmha(lib, b=-1) == 1
    assert call_fmha(lib, d=96) == 2
    assert call_fmha(lib, d=32) == 2
    assert call_fmha(lib, scale=float("nan")) == 1
    assert call_fmha(lib, scale=float("inf")) == 1
    assert call_fmha(lib, scale=-1.0) == 2
    assert call_fmha(lib, mask=_lib.FmhaMask(7, None)) == 2
    assert call_fmha(lib, q=None) == 1
    assert call_fmha(lib, mask=_lib.FmhaMask(1, None)) == 1           # KEY_PADDING needs kv_len
    assert call_fmha(lib, mask=_lib.FmhaMask(3, None, None, 8)) == 1   # KEY_BIAS needs key_bias
    assert call_fmha(lib, mask=_lib.FmhaMask(3, None, 16, 6)) == 1     # stride % 4
    assert call_fmha(lib, mask=_lib.FmhaMask(3, None, 16, 4)) == 1     # stride < seq_kv
    assert call_fmha(lib, mask=_lib.FmhaMask(3, None, 24, 8)) == 3     # misaligned bias
    assert call_fmha(lib, mask=_lib.FmhaMask(3, None, 16, 8), scale=0.0) == 2  # bias / scale needs scale > 0
    assert call_fmha(lib, q=24) == 3                                   # 8-byte aligned only
    assert call_fmha(lib, skv=0) == 1
    # zero work: OK without touching the device
    assert call_fmha(lib, b=0) == 0
    assert call_fmha(lib, sq=0) == 0
    assert call_fmha(lib, q=None, k=None, v=None, o=None, h=0) == 0
    assert lib.gemm_bias_act(16, 16, None, 16, 4, 8, 12, 0, None) == 2  # K % 8
    assert lib.gemm_bias_act(16, 16, None, 16, 4, 8, 16, 9, None) == 2  # act
    assert lib.gemm_bias_act(16, 16, None, 16, 0, 8, 16, 0, None) == 0
    dg = lib.dual_gemm_bias_act
    assert dg(16, 16, 16, 16, None, 16, 4, 8, 16, 12, 1, None) == 2    # K2 % 8
    assert dg(16, 16, 16, 16, None, 16, 4, 8, 16, 16, 5, None) == 2    # act
    assert dg(16, 16, None, 16, None, 16, 4, 8, 16, 16, 1, None) == 1  # null A2
    assert dg(16, 16, 24, 16, None, 16, 4, 8, 16, 16, 1, None) == 3    # misaligned
    assert dg(16, 16, 16, 16, None, 16, 0, 8, 16, 16, 1, None) == 0    # M = 0
    sk = lib.fmha_fwd_splitkv
    assert sk(2, 16, 16, 16, 16, None, 1, 1, 8, 8, 64, 0.1, 2, 16, 1 << 20, None) == 2   # dtype
    assert sk(0, 16, 16, 16, 16, None, 1, 1, 8, 8, 64, 0.1, -1, 16, 1 << 20, None) == 2  # splits
    assert sk(0, 16, 16, 16, 16, None, 1, 1, 8, 8, 96, 0.1, 2, 16, 1 << 20, None) == 2   # head_dim
    assert sk(0, 16, 16, 16, 16, None, 0, 1, 8, 8, 64, 0.1, 2, None, 0, None) == 0       # no work
    assert lib.fmha_splitkv_workspace_bytes(2, 3, 5, 64, 4) == 4 * 2 * 3 * 5 * 66 * 4
    assert lib.fmha_splitkv_workspace_bytes(2, 3, 5, 64, 1) == 0
    mf = lib.mlp_fused_fwd
    assert mf(16, 16, None, 16, 4, 96, 3, 1, None) == 2                # width not 64 / 128
    assert mf(16, 16, None, 16, 4, 128, 0, 1, None) == 2               # no layers
    assert mf(16, 16, None, 16, 4, 128, 3, 9, None) == 2               # act
    assert mf(16, 16, None, 16, -1, 128, 3, 1, None) == 1              # negative M
    assert mf(None, 16, None, 16, 4, 128, 3, 1, None) == 1             # null X
    assert mf(16, 24, None, 16, 4, 128, 3, 1, None) == 3               # misaligned W
    assert mf(None, None, None, None, 0, 128, 3, 1, None) == 0         # M = 0
    # varlen: validation before any device access
    vl = lib.fmha_fwd_varlen
    assert vl(16, 16, 16, 2, 8, 16, 2, 96, 0.1, 0, 0, None) == 2       # head_dim
    assert vl(16, 16, 16, 2, 8, 16, 2, 64, -1.0, 0, 0, None) == 2      # negative scale
    assert vl(16, 16, 16, 2, 8, 16, 2, 64, 0.1, 2, 0, None) == 2       # causal flag
    assert vl(16, 16, 16, 2, 8, 16, 2, 64, 0.1, 0, 5, None) == 2       # dtype
    assert vl(None, 16, 16, 2, 8, 16, 2, 64, 0.1, 0, 0, None) == 1     # null QKV
    assert vl(24, 16, 16, 2, 8, 16, 2, 64, 0.1, 0, 0, None) == 3       # misaligned
    assert vl(16, 16, 16, -1, 8, 16, 2, 64, 0.1, 0, 0, None) == 1
    assert vl(None, None, None, 0, 8, 16, 2, 64, 0.1, 0, 0, None) == 0  # no sequences
    assert lib.fmha_workspace_bytes(2, 3, 100, 50, 64) >= 2 * (2 * 3 * 100 * 64 * 2) + 2 * (2 * 3 * 50 * 64 * 2)


def test_no_device_is_loud(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    # a valid compute call on a machine without an sm_100 device must fail, never fall back
    assert call_fmha(lib) == 5
    assert lib.mlp_fused_fwd(16, 16, None, 16, 4, 128, 3, 1, None) == 5
