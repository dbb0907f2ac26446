"""ctypes binding to libb200fmha.so (the C ABI in include/fmha.h).

Argument marshalling only: every step of the FMHA / GEMM path runs in the CUDA kernels behind
the ABI.  There is no fallback of any kind — a missing library or a non-sm_100 device raises.
"""

from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# B200FMHA_LIB may name another build of the same library (tuning variants under lib/)
LIB_PATH = os.environ.get("B200FMHA_LIB", os.path.join(_HERE, "lib", "libb200fmha.so"))

FMHA_OK = 0
STATUS_NAMES = {
    0: "FMHA_OK",
    1: "FMHA_ERR_INVALID_ARG",
    2: "FMHA_ERR_UNSUPPORTED",
    3: "FMHA_ERR_MISALIGNED",
    4: "FMHA_ERR_CUDA",
    5: "FMHA_ERR_NO_DEVICE",
}

# symbols include/fmha.h declares (tests check every one is exported)
EXPORTED_SYMBOLS = (
    "fmha_fwd",
    "fmha_fwd_bf16",
    "fmha_fwd_strided",
    "fmha_fwd_varlen",
    "fmha_workspace_bytes",
    "fmha_fwd_from_host",
    "fmha_splitkv_default_splits",
    "fmha_splitkv_workspace_bytes",
    "fmha_fwd_splitkv",
    "fmha_fwd_streamk",
    "fmha_streamk_workspace_bytes",
    "fmha_streamk_plan",
    "gemm_bias_act",
    "dual_gemm_bias_act",
    "mlp_fused_fwd",
    "transformer_layer_workspace_bytes",
    "transformer_layer_fwd",
    "fmha_status_string",
    "fmha_last_cuda_error",
    "fmha_version",
)


class FmhaMask(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("kv_len", ctypes.c_void_p), ("key_bias", ctypes.c_void_p),
                ("key_bias_stride", ctypes.c_int32), ("attn_bias", ctypes.c_void_p),
                ("attn_bias_stride_b", ctypes.c_int64), ("attn_bias_stride_h", ctypes.c_int64),
                ("attn_bias_stride_q", ctypes.c_int64)]


class FmhaStrides(ctypes.Structure):
    """fmha_strides_t: element strides {batch, head, row} of Q, K, V, O."""
    _fields_ = [("q", ctypes.c_int64 * 3), ("k", ctypes.c_int64 * 3), ("v", ctypes.c_int64 * 3),
                ("o", ctypes.c_int64 * 3)]


class FmhaError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str = ""):
        self.status = status
        name = STATUS_NAMES.get(status, str(status))
        super().__init__(f"{where} failed: {name}" + (f" ({detail})" if detail else ""))


_lib = None


def load() -> ctypes.CDLL:
    """Load (once) and return the library; raise if it has not been built."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(
            f"{LIB_PATH} not found: build it with `make -C paper_conf_asplos_hagedornfccgg23_b200` "
            "or __graft_entry__.build() (there is no CPU fallback)")
    lib = ctypes.CDLL(LIB_PATH)
    vp, i32, f32, sz = ctypes.c_void_p, ctypes.c_int, ctypes.c_float, ctypes.c_size_t
    mp = ctypes.POINTER(FmhaMask)
    for name in ("fmha_fwd", "fmha_fwd_bf16"):
        f = getattr(lib, name)
        f.argtypes = [vp, vp, vp, vp, mp, i32, i32, i32, i32, i32, f32, vp]
        f.restype = i32
    lib.fmha_fwd_strided.argtypes = [i32, vp, vp, vp, vp, ctypes.POINTER(FmhaStrides), mp, i32, i32, i32, i32, i32,
                                      f32, vp]
    lib.fmha_fwd_strided.restype = i32
    if hasattr(lib, "fmha_fwd_varlen"):  # absent only in old tuning builds (B200FMHA_LIB A/B runs)
        lib.fmha_fwd_varlen.argtypes = [vp, vp, vp, i32, i32, i32, i32, i32, f32, i32, i32, vp]
        lib.fmha_fwd_varlen.restype = i32
    lib.fmha_workspace_bytes.argtypes = [i32] * 5
    lib.fmha_workspace_bytes.restype = sz
    lib.fmha_fwd_from_host.argtypes = [i32, vp, vp, vp, vp, mp, vp, sz, i32, i32, i32, i32, i32, f32, vp]
    lib.fmha_fwd_from_host.restype = i32
    lib.gemm_bias_act.argtypes = [vp, vp, vp, vp, i32, i32, i32, i32, vp]
    lib.gemm_bias_act.restype = i32
    if hasattr(lib, "fmha_fwd_splitkv"):
        lib.fmha_splitkv_default_splits.argtypes = [i32] * 4
        lib.fmha_splitkv_default_splits.restype = i32
        lib.fmha_splitkv_workspace_bytes.argtypes = [i32] * 5
        lib.fmha_splitkv_workspace_bytes.restype = sz
        lib.fmha_fwd_splitkv.argtypes = [i32, vp, vp, vp, vp, mp, i32, i32, i32, i32, i32, f32, i32, vp, sz, vp]
        lib.fmha_fwd_splitkv.restype = i32
    if hasattr(lib, "fmha_fwd_streamk"):  # absent only in old tuning builds
        lib.fmha_fwd_streamk.argtypes = [i32, vp, vp, vp, vp, mp, i32, i32, i32, i32, i32, f32, vp, sz, vp]
        lib.fmha_fwd_streamk.restype = i32
        lib.fmha_streamk_workspace_bytes.argtypes = [i32, i32]
        lib.fmha_streamk_workspace_bytes.restype = sz
        lib.fmha_streamk_plan.argtypes = [i32, i32, i32, i32, i32, i32, ctypes.POINTER(i32)]
        lib.fmha_streamk_plan.restype = i32
    if hasattr(lib, "mlp_fused_fwd"):
        lib.mlp_fused_fwd.argtypes = [vp, vp, vp, vp, i32, i32, i32, i32, vp]
        lib.mlp_fused_fwd.restype = i32
    if hasattr(lib, "dual_gemm_bias_act"):
        lib.dual_gemm_bias_act.argtypes = [vp, vp, vp, vp, vp, vp, i32, i32, i32, i32, i32, vp]
        lib.dual_gemm_bias_act.restype = i32
    if hasattr(lib, "transformer_layer_fwd"):  # absent only in old tuning builds
        lib.transformer_layer_workspace_bytes.argtypes = [i32, i32, i32]
        lib.transformer_layer_workspace_bytes.restype = sz
        lib.transformer_layer_fwd.argtypes = [vp] * 10 + [vp, i32, i32, i32, i32, i32, i32, f32, i32, vp, sz, vp]
        lib.transformer_layer_fwd.restype = i32
    for name in ("fmha_status_string",):
        getattr(lib, name).argtypes = [i32]
        getattr(lib, name).restype = ctypes.c_char_p
    lib.fmha_last_cuda_error.argtypes = []
    lib.fmha_last_cuda_error.restype = ctypes.c_char_p
    lib.fmha_version.argtypes = []
    lib.fmha_version.restype = ctypes.c_char_p
    _lib = lib
    return lib


def check(status: int, where: str) -> None:
    if status != FMHA_OK:
        detail = load().fmha_last_cuda_error().decode() if status == 4 else ""
        raise FmhaError(status, where, detail)
