"""B200-native (sm_100a) fused multi-head attention forward and GEMM+bias+activation.

Python surface over the C ABI of ``lib/libb200fmha.so`` (include/fmha.h).  PyTorch provides
device memory and streams only; every step of the computation runs in the hand-written CUDA
kernels behind the ABI.  There is no CPU or library fallback: without the built library or an
sm_100 device these functions raise.

    fmha_fwd(q, k, v, kv_len=None, causal=False, scale=None, out=None) -> O
    fmha_fwd_varlen(qkv, cu_seqlens, max_seqlen, causal=False, scale=None, out=None) -> O
    fmha_fwd_from_host(q, k, v, ..., workspace) -> O  (host tensors; copies inside the call)
    gemm_bias_act(a, w, bias=None, act="none", out=None) -> C
    dual_gemm_bias_act(a1, w1, a2, w2, bias=None, act="relu", out=None) -> C  (simplified LSTM cell)
    transformer_layer(x, weights, cu_seqlens, max_seqlen, heads, ...) -> Y  (5 launches, one call)
"""

from __future__ import annotations

import ctypes
import math

import torch

from . import _lib
from ._lib import FmhaError, FmhaMask, FmhaStrides

__all__ = ["fmha_fwd", "fmha_fwd_splitkv", "fmha_fwd_streamk", "streamk_plan", "fmha_fwd_varlen", "fmha_fwd_from_host", "gemm_bias_act", "dual_gemm_bias_act", "mlp_fused", "transformer_layer", "layer_workspace_bytes", "workspace_bytes", "FmhaError",
           "MASK_NONE", "MASK_KEY_PADDING", "MASK_CAUSAL", "MASK_KEY_BIAS", "MASK_ATTN_BIAS", "ACTS", "version"]

MASK_NONE, MASK_KEY_PADDING, MASK_CAUSAL, MASK_KEY_BIAS, MASK_ATTN_BIAS = 0, 1, 2, 3, 4
ACTS = {"none": 0, "relu": 1, "gelu": 2, "gelu_erf": 2, "gelu_tanh": 3, "tanh": 4}


def version() -> str:
    return _lib.load().fmha_version().decode()


def _stream_ptr(dev: torch.device) -> int:
    return torch.cuda.current_stream(dev).cuda_stream


def _check_out(out: torch.Tensor, shape, dtype, like: torch.Tensor, what: str) -> None:
    """A caller-supplied output must be exactly what the kernel writes: shape, dtype, dense
    row-major layout and the inputs' device (the kernels write every element through raw pointers)."""
    if tuple(out.shape) != tuple(shape) or out.dtype != dtype or not out.is_contiguous() or out.device != like.device:
        raise ValueError(f"{what}: out must be a contiguous {dtype} tensor of shape {tuple(shape)} on {like.device}, "
                         f"got {out.dtype} {tuple(out.shape)} on {out.device}")


def _check_bias(bias: torch.Tensor | None, shape, like: torch.Tensor, what: str) -> torch.Tensor | None:
    """Bias vectors are read for every output column: exact shape, fp16, on the inputs' device; the
    contiguous copy is returned so the caller keeps it alive across the launch."""
    if bias is None:
        return None
    if tuple(bias.shape) != tuple(shape) or bias.dtype != torch.float16 or bias.device != like.device:
        raise ValueError(f"{what}: bias must be fp16 {tuple(shape)} on {like.device}, got {bias.dtype} "
                         f"{tuple(bias.shape)} on {bias.device}")
    return bias.contiguous()


def _mask(kv_len, causal: bool):
    if kv_len is not None and causal:
        raise ValueError("key padding and causal masks are mutually exclusive in this ABI")
    if kv_len is not None:
        return FmhaMask(MASK_KEY_PADDING, kv_len.data_ptr())
    if causal:
        return FmhaMask(MASK_CAUSAL, None)
    return FmhaMask(MASK_NONE, None)


def _bhsd_strides(t: torch.Tensor, what: str):
    """{batch, head, row} element strides of a [B, H, S, D] view whose last dimension is contiguous."""
    if t.dim() != 4 or t.stride(3) != 1:
        raise ValueError(f"{what} must be a 4-D [B,H,S,D] view with head_dim contiguous (stride 1)")
    st = (t.stride(0), t.stride(1), t.stride(2))
    # size-1 dimensions may carry any stride; give them a legal one for the tensor map
    st = tuple(s if t.shape[i] > 1 else max(8, t.shape[3]) * max(1, t.shape[2]) for i, s in enumerate(st))
    if any(s % 8 for s in st):
        raise ValueError(f"{what}: strides must be multiples of 8 elements (16 bytes, TMA), got {st}")
    return st


def fmha_fwd(q: torch.Tensor, k: torch.Tensor, v: torch.Tensor, kv_len: torch.Tensor | None = None,
             causal: bool = False, scale: float | None = None, out: torch.Tensor | None = None,
             key_bias: torch.Tensor | None = None, attn_bias: torch.Tensor | None = None) -> torch.Tensor:
    """O = softmax(scale * Q K^T + mask) V.  q: [B,H,Sq,D], k/v: [B,H,Skv,D] CUDA fp16/bf16 tensors
    (any strides with head_dim contiguous and the others multiples of 8 elements -- e.g. a [B,S,H,D]
    tensor viewed with .transpose(1, 2); non-contiguous views go through ``fmha_fwd_strided``);
    kv_len: CUDA int32 [B] (key padding) or None; causal: bottom-right mask; key_bias: CUDA fp32
    [B, stride >= Skv] additive per-key bias (stride % 4 == 0; -inf excludes a key); attn_bias: a CUDA
    tensor of q's dtype broadcastable to [B, H, Sq, Skv] (additive (query x key) mask, R21;
    its last dimension contiguous, row stride a multiple of 8 and >= Skv).  The mask kinds are
    exclusive.  Calls ``fmha_fwd`` / ``fmha_fwd_bf16`` / ``fmha_fwd_strided`` of the C ABI on the
    current stream."""
    lib = _lib.load()
    if q.dtype not in (torch.float16, torch.bfloat16) or k.dtype != q.dtype or v.dtype != q.dtype:
        raise TypeError("q, k, v must share dtype fp16 or bf16")
    if not (q.is_cuda and k.is_cuda and v.is_cuda):
        raise TypeError("q, k, v must be CUDA tensors (no CPU fallback)")
    if q.dim() != 4:
        raise ValueError("q, k, v must be 4-D [B,H,S,D]")
    b, h, sq, d = q.shape
    skv = k.shape[2]
    if k.shape != (b, h, skv, d) or v.shape != k.shape:
        raise ValueError(f"shape mismatch q{tuple(q.shape)} k{tuple(k.shape)} v{tuple(v.shape)}")
    if kv_len is not None:
        if kv_len.dtype != torch.int32 or not kv_len.is_cuda or kv_len.numel() != b:
            raise ValueError("kv_len must be a CUDA int32 tensor of length batch")
        kv_len = kv_len.contiguous()
    if out is None:
        out = torch.empty((b, h, sq, d), dtype=q.dtype, device=q.device)
    elif tuple(out.shape) != (b, h, sq, d) or out.dtype != q.dtype or out.device != q.device:
        raise ValueError("out must be a [B,H,Sq,D] tensor of q's dtype on q's device")
    scale = 1.0 / math.sqrt(d) if scale is None else float(scale)
    kinds = sum(x is not None and x is not False for x in (kv_len, causal or None, key_bias, attn_bias))
    if kinds > 1:
        raise ValueError("kv_len, causal, key_bias and attn_bias are exclusive")
    if key_bias is not None:
        if key_bias.dtype != torch.float32 or not key_bias.is_cuda or key_bias.dim() != 2 or key_bias.shape[0] != b:
            raise ValueError("key_bias must be a CUDA float32 tensor [batch, stride]")
        if key_bias.stride(1) != 1:
            raise ValueError("key_bias rows must be contiguous")
        m = FmhaMask(MASK_KEY_BIAS, None, key_bias.data_ptr(), key_bias.stride(0))
    elif attn_bias is not None:
        if attn_bias.dtype != q.dtype or not attn_bias.is_cuda or attn_bias.device != q.device:
            raise ValueError("attn_bias must be a CUDA tensor of q's dtype on q's device")
        ab = attn_bias
        while ab.dim() < 4:
            ab = ab.unsqueeze(0)
        ab = ab.expand(b, h, sq, skv)  # broadcast dimensions get stride 0
        if ab.stride(3) != 1 or ab.stride(2) % 8 or 0 < ab.stride(2) < skv or (ab.stride(2) == 0 and skv % 8):
            raise ValueError("attn_bias rows must be contiguous with a row stride >= Skv and a multiple of 8 "
                             "(or 0, broadcast over queries, with Skv a multiple of 8)")
        m = FmhaMask(MASK_ATTN_BIAS, None, None, 0, ab.data_ptr(), ab.stride(0), ab.stride(1), ab.stride(2))
    else:
        m = _mask(kv_len, causal)
    st = _stream_ptr(q.device)
    if all(t.is_contiguous() for t in (q, k, v, out)):
        fn = lib.fmha_fwd if q.dtype == torch.float16 else lib.fmha_fwd_bf16
        status = fn(q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(), ctypes.byref(m), b, h, sq, skv, d,
                    scale, st)
        _lib.check(status, "fmha_fwd")
        return out
    strides = FmhaStrides((ctypes.c_int64 * 3)(*_bhsd_strides(q, "q")), (ctypes.c_int64 * 3)(*_bhsd_strides(k, "k")),
                          (ctypes.c_int64 * 3)(*_bhsd_strides(v, "v")), (ctypes.c_int64 * 3)(*_bhsd_strides(out, "out")))
    status = lib.fmha_fwd_strided(0 if q.dtype == torch.float16 else 1, q.data_ptr(), k.data_ptr(), v.data_ptr(),
                                  out.data_ptr(), ctypes.byref(strides), ctypes.byref(m), b, h, sq, skv, d, scale, st)
    _lib.check(status, "fmha_fwd_strided")
    return out


def fmha_fwd_splitkv(q: torch.Tensor, k: torch.Tensor, v: torch.Tensor, kv_len: torch.Tensor | None = None,
                     causal: bool = False, scale: float | None = None, num_splits: int = 0,
                     out: torch.Tensor | None = None, workspace: torch.Tensor | None = None) -> torch.Tensor:
    """The same operation as fmha_fwd with each row's keys split over `num_splits` work items and
    merged by a second kernel (0 = the library's default for this shape).  `workspace` (a CUDA byte
    tensor) is allocated here when not given.  Calls ``fmha_fwd_splitkv`` of the C ABI."""
    lib = _lib.load()
    if q.dtype not in (torch.float16, torch.bfloat16) or k.dtype != q.dtype or v.dtype != q.dtype:
        raise TypeError("q, k, v must share dtype fp16 or bf16")
    if not (q.is_cuda and k.is_cuda and v.is_cuda):
        raise TypeError("q, k, v must be CUDA tensors (no CPU fallback)")
    if not (q.is_contiguous() and k.is_contiguous() and v.is_contiguous()):
        raise ValueError("q, k, v must be contiguous [B,H,S,D]")
    b, h, sq, d = q.shape
    skv = k.shape[2]
    if k.shape != (b, h, skv, d) or v.shape != k.shape:
        raise ValueError(f"shape mismatch q{tuple(q.shape)} k{tuple(k.shape)} v{tuple(v.shape)}")
    if kv_len is not None:
        if kv_len.dtype != torch.int32 or not kv_len.is_cuda or kv_len.numel() != b:
            raise ValueError("kv_len must be a CUDA int32 tensor of length batch")
        kv_len = kv_len.contiguous()
    if out is None:
        out = torch.empty_like(q)
    else:
        _check_out(out, q.shape, q.dtype, q, "fmha_fwd_splitkv")
    splits = num_splits if num_splits > 0 else lib.fmha_splitkv_default_splits(b, h, sq, skv)
    need = lib.fmha_splitkv_workspace_bytes(b, h, sq, d, splits)
    if workspace is None or workspace.numel() < need:
        workspace = torch.empty(max(need, 16), dtype=torch.uint8, device=q.device)
    scale = 1.0 / math.sqrt(d) if scale is None else float(scale)
    m = _mask(kv_len, causal)
    st = lib.fmha_fwd_splitkv(0 if q.dtype == torch.float16 else 1, q.data_ptr(), k.data_ptr(), v.data_ptr(),
                              out.data_ptr(), ctypes.byref(m), b, h, sq, skv, d, scale, splits,
                              workspace.data_ptr(), workspace.numel(), _stream_ptr(q.device))
    _lib.check(st, "fmha_fwd_splitkv")
    return out


_STREAMK_WS: dict = {}


def streamk_workspace(device: torch.device, head_dim: int) -> torch.Tensor:
    """The zero-filled workspace of fmha_fwd_streamk for `device` and its current stream (cached per
    (device, head_dim, stream): every launch leaves it zero-filled again, so one buffer serves all
    launches on one stream; launches on different streams get different buffers, since two concurrent
    launches must not share the per-item counters)."""
    lib = _lib.load()
    device = torch.device(device)
    dev_index = device.index if device.index is not None else torch.cuda.current_device()
    key = (dev_index, head_dim, torch.cuda.current_stream(dev_index).cuda_stream)
    ws = _STREAMK_WS.get(key)
    if ws is None:
        with torch.cuda.device(device):
            need = lib.fmha_streamk_workspace_bytes(head_dim, 0)
        if need == 0:
            raise RuntimeError("fmha_streamk_workspace_bytes: no sm_100 device or unsupported head_dim")
        ws = torch.zeros(need, dtype=torch.uint8, device=device)
        _STREAMK_WS[key] = ws
    return ws


def streamk_plan(batch: int, heads: int, seq_q: int, seq_kv: int, sm_count: int,
                 mask_kind: int = 0) -> tuple[int, int]:
    """(key splits of each last-round item, items in the last round) of fmha_fwd_streamk's schedule
    on a GPU with `sm_count` SMs (host-only; ``fmha_streamk_plan`` of the C ABI)."""
    lib = _lib.load()
    tail = ctypes.c_int(0)
    s = lib.fmha_streamk_plan(batch, heads, seq_q, seq_kv, mask_kind, sm_count, ctypes.byref(tail))
    return s, tail.value


def fmha_fwd_streamk(q: torch.Tensor, k: torch.Tensor, v: torch.Tensor, kv_len: torch.Tensor | None = None,
                     causal: bool = False, scale: float | None = None, out: torch.Tensor | None = None,
                     workspace: torch.Tensor | None = None) -> torch.Tensor:
    """fmha_fwd in one launch whose last, partial round of work items is split along the keys and
    merged in the kernel by the piece that finishes last (stream-K tail).  q, k, v contiguous
    [B,H,S,D] CUDA fp16/bf16.  `workspace` defaults to a cached zero-filled per-device buffer.  Calls
    ``fmha_fwd_streamk`` of the C ABI."""
    lib = _lib.load()
    if q.dtype not in (torch.float16, torch.bfloat16) or k.dtype != q.dtype or v.dtype != q.dtype:
        raise TypeError("q, k, v must share dtype fp16 or bf16")
    if not (q.is_cuda and k.is_cuda and v.is_cuda):
        raise TypeError("q, k, v must be CUDA tensors (no CPU fallback)")
    if not (q.is_contiguous() and k.is_contiguous() and v.is_contiguous()):
        raise ValueError("q, k, v must be contiguous [B,H,S,D]")
    b, h, sq, d = q.shape
    skv = k.shape[2]
    if k.shape != (b, h, skv, d) or v.shape != k.shape:
        raise ValueError(f"shape mismatch q{tuple(q.shape)} k{tuple(k.shape)} v{tuple(v.shape)}")
    if kv_len is not None:
        if kv_len.dtype != torch.int32 or not kv_len.is_cuda or kv_len.numel() != b:
            raise ValueError("kv_len must be a CUDA int32 tensor of length batch")
        kv_len = kv_len.contiguous()
    if out is None:
        out = torch.empty_like(q)
    else:
        _check_out(out, q.shape, q.dtype, q, "fmha_fwd_streamk")
    if workspace is None:
        workspace = streamk_workspace(q.device, d)
    scale = 1.0 / math.sqrt(d) if scale is None else float(scale)
    m = _mask(kv_len, causal)
    st = lib.fmha_fwd_streamk(0 if q.dtype == torch.float16 else 1, q.data_ptr(), k.data_ptr(), v.data_ptr(),
                              out.data_ptr(), ctypes.byref(m), b, h, sq, skv, d, scale, workspace.data_ptr(),
                              workspace.numel(), _stream_ptr(q.device))
    _lib.check(st, "fmha_fwd_streamk")
    return out


def fmha_fwd_varlen(qkv: torch.Tensor, cu_seqlens: torch.Tensor, max_seqlen: int, causal: bool = False,
                    scale: float | None = None, out: torch.Tensor | None = None) -> torch.Tensor:
    """Packed variable-length FMHA (MLPerf BERT layout): qkv [T,3,H,D] contiguous CUDA fp16/bf16,
    cu_seqlens CUDA int32 [num_seqs+1] (sequence s = tokens cu[s]..cu[s+1]-1), max_seqlen a host
    int >= every length.  Returns O [T,H,D].  Calls ``fmha_fwd_varlen`` of the C ABI."""
    lib = _lib.load()
    if qkv.dtype not in (torch.float16, torch.bfloat16):
        raise TypeError("qkv must be fp16 or bf16")
    if not qkv.is_cuda or not cu_seqlens.is_cuda:
        raise TypeError("qkv and cu_seqlens must be CUDA tensors (no CPU fallback)")
    if qkv.dim() != 4 or qkv.shape[1] != 3 or not qkv.is_contiguous():
        raise ValueError("qkv must be contiguous [T,3,H,D]")
    if cu_seqlens.dtype != torch.int32 or cu_seqlens.dim() != 1 or cu_seqlens.numel() < 1:
        raise ValueError("cu_seqlens must be a CUDA int32 tensor [num_seqs+1]")
    t, _, h, d = qkv.shape
    cu_seqlens = cu_seqlens.contiguous()
    if out is None:
        out = torch.empty((t, h, d), dtype=qkv.dtype, device=qkv.device)
    elif out.shape != (t, h, d) or out.dtype != qkv.dtype or not out.is_contiguous():
        raise ValueError("out must be contiguous [T,H,D] of qkv's dtype")
    scale = 1.0 / math.sqrt(d) if scale is None else float(scale)
    st = lib.fmha_fwd_varlen(qkv.data_ptr(), out.data_ptr(), cu_seqlens.data_ptr(), cu_seqlens.numel() - 1,
                             int(max_seqlen), t, h, d, scale, int(bool(causal)),
                             0 if qkv.dtype == torch.float16 else 1, _stream_ptr(qkv.device))
    _lib.check(st, "fmha_fwd_varlen")
    return out


def workspace_bytes(b: int, h: int, sq: int, skv: int, d: int) -> int:
    return int(_lib.load().fmha_workspace_bytes(b, h, sq, skv, d))


def fmha_fwd_from_host(q: torch.Tensor, k: torch.Tensor, v: torch.Tensor, out: torch.Tensor,
                       workspace: torch.Tensor, kv_len: torch.Tensor | None = None, causal: bool = False,
                       scale: float | None = None, stream: torch.cuda.Stream | None = None) -> torch.Tensor:
    """End-to-end call with HOST (pinned) q/k/v/out and a device workspace: H2D copies, kernel and
    D2H copy are ordered after ``stream``'s queued work and joined back into it by ``fmha_fwd_from_host`` of the C ABI (async; the
    caller synchronises before reading ``out``)."""
    lib = _lib.load()
    if q.dtype not in (torch.float16, torch.bfloat16) or k.dtype != q.dtype or v.dtype != q.dtype or out.dtype != q.dtype:
        raise TypeError("q, k, v, out must share dtype fp16 or bf16")
    if any(t.is_cuda for t in (q, k, v, out)):
        raise TypeError("fmha_fwd_from_host takes HOST q, k, v, out (use fmha_fwd for device tensors)")
    if not all(t.is_contiguous() for t in (q, k, v, out)):
        raise ValueError("q, k, v, out must be contiguous [B,H,S,D]")
    if not workspace.is_cuda:
        raise TypeError("workspace must be a CUDA tensor")
    b, h, sq, d = q.shape
    skv = k.shape[2]
    if k.shape != (b, h, skv, d) or v.shape != k.shape or out.shape != q.shape:
        raise ValueError(f"shape mismatch q{tuple(q.shape)} k{tuple(k.shape)} v{tuple(v.shape)} out{tuple(out.shape)}")
    if kv_len is not None and (kv_len.is_cuda or kv_len.dtype != torch.int32 or kv_len.numel() != b
                               or not kv_len.is_contiguous()):
        raise ValueError("kv_len must be a contiguous HOST int32 tensor of length batch for fmha_fwd_from_host")
    dt = {torch.float16: 0, torch.bfloat16: 1}[q.dtype]
    m = FmhaMask(MASK_NONE, None)
    if kv_len is not None:
        m = FmhaMask(MASK_KEY_PADDING, kv_len.data_ptr())  # HOST int32 for this entry point
    elif causal:
        m = FmhaMask(MASK_CAUSAL, None)
    scale = 1.0 / math.sqrt(d) if scale is None else float(scale)
    s = stream if stream is not None else torch.cuda.current_stream(workspace.device)
    st = lib.fmha_fwd_from_host(dt, q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(), ctypes.byref(m),
                                workspace.data_ptr(), workspace.numel() * workspace.element_size(), b, h, sq, skv,
                                d, scale, s.cuda_stream)
    _lib.check(st, "fmha_fwd_from_host")
    return out


def gemm_bias_act(a: torch.Tensor, w: torch.Tensor, bias: torch.Tensor | None = None, act: str = "none",
                  out: torch.Tensor | None = None) -> torch.Tensor:
    """C = act(A W^T + bias): a [M,K], w [N,K], bias [N] fp16 CUDA tensors -> [M,N] fp16."""
    lib = _lib.load()
    if a.dtype != torch.float16 or w.dtype != torch.float16 or (bias is not None and bias.dtype != torch.float16):
        raise TypeError("gemm_bias_act takes fp16 tensors")
    if not (a.is_cuda and w.is_cuda):
        raise TypeError("CUDA tensors required (no CPU fallback)")
    a, w = a.contiguous(), w.contiguous()
    m_, k_ = a.shape
    n_ = w.shape[0]
    if w.shape[1] != k_:
        raise ValueError("K mismatch")
    bias = _check_bias(bias, (n_,), a, "gemm_bias_act")
    if out is None:
        out = torch.empty((m_, n_), dtype=torch.float16, device=a.device)
    else:
        _check_out(out, (m_, n_), torch.float16, a, "gemm_bias_act")
    st = lib.gemm_bias_act(a.data_ptr(), w.data_ptr(), None if bias is None else bias.data_ptr(),
                           out.data_ptr(), m_, n_, k_, ACTS[act], _stream_ptr(a.device))
    _lib.check(st, "gemm_bias_act")
    return out


def layer_workspace_bytes(tokens: int, d_model: int, d_ff: int) -> int:
    return int(_lib.load().transformer_layer_workspace_bytes(tokens, d_model, d_ff))


def transformer_layer(x: torch.Tensor, wqkv: torch.Tensor, bqkv, wo: torch.Tensor, bo, w1: torch.Tensor, b1,
                      w2: torch.Tensor, b2, cu_seqlens: torch.Tensor, max_seqlen: int, heads: int,
                      causal: bool = False, scale: float | None = None, out: torch.Tensor | None = None,
                      workspace: torch.Tensor | None = None) -> torch.Tensor:
    """Y = MLP(out_proj(FMHA(QKV_proj(x)))) for packed tokens x [T, d_model] (fp16 CUDA), one call to
    ``transformer_layer_fwd`` of the C ABI (R18).  Weights in nn.Linear layout [out, in];
    biases [out] or None."""
    lib = _lib.load()
    ts = [x, wqkv, wo, w1, w2] + [b for b in (bqkv, bo, b1, b2) if b is not None]
    if any(t.dtype != torch.float16 or not t.is_cuda or not t.is_contiguous() for t in ts):
        raise TypeError("transformer_layer takes contiguous fp16 CUDA tensors")
    t_, d = x.shape
    d_ff = w1.shape[0]
    if wqkv.shape != (3 * d, d) or wo.shape != (d, d) or w1.shape != (d_ff, d) or w2.shape != (d, d_ff):
        raise ValueError("weight shapes must be Wqkv [3d,d], Wo [d,d], W1 [d_ff,d], W2 [d,d_ff]")
    if cu_seqlens.dtype != torch.int32 or not cu_seqlens.is_cuda:
        raise ValueError("cu_seqlens must be a CUDA int32 tensor")
    if out is None:
        out = torch.empty((t_, d), dtype=torch.float16, device=x.device)
    need = layer_workspace_bytes(t_, d, d_ff)
    if workspace is None or workspace.numel() * workspace.element_size() < need:
        workspace = torch.empty(need, dtype=torch.uint8, device=x.device)
    scale = 1.0 / math.sqrt(d // heads) if scale is None else float(scale)
    ptr = lambda b: None if b is None else b.data_ptr()
    st = lib.transformer_layer_fwd(x.data_ptr(), wqkv.data_ptr(), ptr(bqkv), wo.data_ptr(), ptr(bo), w1.data_ptr(),
                                   ptr(b1), w2.data_ptr(), ptr(b2), out.data_ptr(), cu_seqlens.data_ptr(),
                                   cu_seqlens.numel() - 1, int(max_seqlen), t_, d, heads, d_ff, scale,
                                   int(bool(causal)), workspace.data_ptr(),
                                   workspace.numel() * workspace.element_size(), _stream_ptr(x.device))
    _lib.check(st, "transformer_layer_fwd")
    return out


def dual_gemm_bias_act(a1: torch.Tensor, w1: torch.Tensor, a2: torch.Tensor, w2: torch.Tensor,
                       bias: torch.Tensor | None = None, act: str = "relu",
                       out: torch.Tensor | None = None) -> torch.Tensor:
    """C = act(A1 W1^T + A2 W2^T + bias) in one kernel (the paper's simplified LSTM cell, Fig. 12):
    a1 [M,K1], w1 [N,K1], a2 [M,K2], w2 [N,K2], bias [N]; fp16 CUDA tensors -> [M,N] fp16."""
    lib = _lib.load()
    ts = [a1, w1, a2, w2] + ([] if bias is None else [bias])
    if any(t.dtype != torch.float16 or not t.is_cuda for t in ts):
        raise TypeError("dual_gemm_bias_act takes fp16 CUDA tensors (no CPU fallback)")
    a1, w1, a2, w2 = (t.contiguous() for t in (a1, w1, a2, w2))
    m_, k1 = a1.shape
    n_, k2 = w1.shape[0], a2.shape[1]
    if w1.shape[1] != k1 or a2.shape[0] != m_ or w2.shape != (n_, k2):
        raise ValueError("shape mismatch")
    bias = _check_bias(bias, (n_,), a1, "dual_gemm_bias_act")
    if out is None:
        out = torch.empty((m_, n_), dtype=torch.float16, device=a1.device)
    else:
        _check_out(out, (m_, n_), torch.float16, a1, "dual_gemm_bias_act")
    st = lib.dual_gemm_bias_act(a1.data_ptr(), w1.data_ptr(), a2.data_ptr(), w2.data_ptr(),
                                None if bias is None else bias.data_ptr(), out.data_ptr(),
                                m_, n_, k1, k2, ACTS[act], _stream_ptr(a1.device))
    _lib.check(st, "dual_gemm_bias_act")
    return out


def mlp_fused(x: torch.Tensor, w: torch.Tensor, bias: torch.Tensor | None = None, act: str = "relu",
              out: torch.Tensor | None = None) -> torch.Tensor:
    """Y = h_L of h_l = act(h_{l-1} W_l^T + b_l) in ONE kernel (the paper's fused multi-layer MLP,
    Fig. 11): x [M,N], w [L,N,N], bias [L,N]; N in {64, 128}; fp16 CUDA tensors -> [M,N] fp16."""
    lib = _lib.load()
    ts = [x, w] + ([] if bias is None else [bias])
    if any(t.dtype != torch.float16 or not t.is_cuda for t in ts):
        raise TypeError("mlp_fused takes fp16 CUDA tensors (no CPU fallback)")
    x, w = x.contiguous(), w.contiguous()
    m_, n_ = x.shape
    layers = w.shape[0]
    if w.shape != (layers, n_, n_) or (bias is not None and bias.shape != (layers, n_)):
        raise ValueError("shape mismatch")
    bias = _check_bias(bias, (layers, n_), x, "mlp_fused")
    if out is None:
        out = torch.empty((m_, n_), dtype=torch.float16, device=x.device)
    else:
        _check_out(out, (m_, n_), torch.float16, x, "mlp_fused")
    st = lib.mlp_fused_fwd(x.data_ptr(), w.data_ptr(), None if bias is None else bias.data_ptr(),
                           out.data_ptr(), m_, n_, layers, ACTS[act], _stream_ptr(x.device))
    _lib.check(st, "mlp_fused_fwd")
    return out
