"""Seeded synthetic workloads shared by the tests, the bench and smoke().

This module holds NONE of the method's arithmetic: it only defines the shapes of
BASELINE.json's configs and draws seeded random inputs, rounded (RNE) to the I/O
dtype.  Both the CUDA path and the oracle consume what it produces; neither is
imported here.

Recipe:
  * seed 20230325 (the paper's conference date); every (b, h) slice of every
    tensor is drawn from its own ``SeedSequence([seed, cfg_id, tensor_id, b, h])``
    so a shard (a contiguous range of b) reproduces the global tensor exactly;
  * Q, K ~ N(0, 1) (scaled scores ~ N(0, 1) at scale = 1/sqrt(D)); V ~ U(-1, 1),
    so |O| <= 1; the stress variant draws Q, K ~ N(0, 3^2);
  * drawn in float32, then rounded to fp16 / bf16 with round-to-nearest-even;
  * key padding (BERT-base config): kv_len[b] ~ U{32..S}, with kv_len[0] = S so
    at least one batch is unpadded;
  * MLP: A ~ U(-1, 1), W ~ N(0, 1/K), b ~ U(-1, 1);
  * packed variable-length batches (MLPerf BERT inference layout):
    sequence lengths ~ round(N(175, 75^2)) clipped to [32, max_seqlen], with
    sequence 0 at max_seqlen (SQuAD v1.1 tokenised for MLPerf BERT averages ~170
    tokens with a 384 cap -- an assumption); Q, K, V of each
    (sequence, head) drawn like the dense configs' (b, h) slices.
"""

from __future__ import annotations

from dataclasses import dataclass, replace

import numpy as np
import torch

SEED = 20230325

MASK_NONE, MASK_KEY_PADDING, MASK_CAUSAL = 0, 1, 2


@dataclass(frozen=True)
class FmhaConfig:
    name: str
    cfg_id: int
    batch: int
    heads: int
    seq_q: int
    seq_kv: int
    head_dim: int
    dtype: str          # "fp16" | "bf16"
    mask: int = MASK_NONE
    qk_sigma: float = 1.0

    @property
    def units(self) -> int:
        return self.batch * self.heads

    @property
    def scale(self) -> float:
        return float(np.float32(1.0 / np.sqrt(self.head_dim)))

    @property
    def torch_dtype(self):
        return torch.float16 if self.dtype == "fp16" else torch.bfloat16

    def with_(self, **kw) -> "FmhaConfig":
        return replace(self, **kw)


# BASELINE.json "configs" (BJ:L7-L11)
CONFIGS = {
    "tiny": FmhaConfig("tiny", 1, 1, 1, 64, 64, 64, "fp16"),
    "bert_base_pad": FmhaConfig("bert_base_pad", 2, 32, 12, 128, 128, 64, "fp16", MASK_KEY_PADDING),
    "bert_large_384": FmhaConfig("bert_large_384", 3, 32, 16, 384, 384, 64, "fp16"),
    "bert_large_512": FmhaConfig("bert_large_512", 4, 32, 16, 512, 512, 64, "fp16"),
    "gpt_causal": FmhaConfig("gpt_causal", 5, 8, 32, 2048, 2048, 128, "bf16", MASK_CAUSAL),
}


# split-KV: few (b, h) units, a short query block, long keys -- the shape where one
# work item per (b, h, q-tile pair) leaves most SMs idle (decode / speculative-decode blocks)
SPLITKV_CONFIGS = {
    "decode_splitkv": FmhaConfig("decode_splitkv", 14, 4, 8, 16, 16384, 128, "bf16"),
}


@dataclass(frozen=True)
class MlpConfig:
    name: str
    cfg_id: int
    tokens: int
    d_model: int
    d_ff: int
    dtype: str = "fp16"


MLP_CONFIG = MlpConfig("mlp", 6, 16384, 1024, 4096)


@dataclass(frozen=True)
class VarlenConfig:
    """A packed variable-length batch: QKV [T, 3, H, D], cu_seqlens [num_seqs + 1]."""
    name: str
    cfg_id: int
    num_seqs: int
    heads: int
    max_seqlen: int
    head_dim: int
    dtype: str = "fp16"
    causal: bool = False
    mean_len: float = 175.0
    sd_len: float = 75.0
    min_len: int = 32

    @property
    def scale(self) -> float:
        return float(np.float32(1.0 / np.sqrt(self.head_dim)))

    @property
    def torch_dtype(self):
        return torch.float16 if self.dtype == "fp16" else torch.bfloat16

    def with_(self, **kw) -> "VarlenConfig":
        return replace(self, **kw)


# MLPerf-style BERT-large inference batch (the paper's workload): 32 sequences, 16 heads,
# D = 64, max 384 tokens, packed without padding
VARLEN_CONFIGS = {
    "bert_large_varlen": VarlenConfig("bert_large_varlen", 8, 32, 16, 384, 64),
}


def varlen_lengths(cfg: VarlenConfig, seq_offset: int = 0, seed: int = SEED) -> np.ndarray:
    out = np.empty(cfg.num_seqs, dtype=np.int64)
    for s in range(cfg.num_seqs):
        gs = s + seq_offset
        if gs == 0:
            out[s] = cfg.max_seqlen
        else:
            x = _rng(cfg.cfg_id, 9, gs, 0, seed).normal(cfg.mean_len, cfg.sd_len)
            out[s] = int(np.clip(np.rint(x), min(cfg.min_len, cfg.max_seqlen), cfg.max_seqlen))
    return out


def make_varlen_inputs(cfg: VarlenConfig, seq_offset: int = 0, seed: int = SEED, lengths=None):
    """Returns (qkv [T,3,H,D] CPU tensor in cfg's dtype, cu_seqlens int32 numpy [num_seqs+1]).
    Global sequence index = s + seq_offset.  ``lengths`` overrides the drawn lengths."""
    lens = varlen_lengths(cfg, seq_offset, seed) if lengths is None else np.asarray(lengths, dtype=np.int64)
    cu = np.zeros(len(lens) + 1, dtype=np.int32)
    cu[1:] = np.cumsum(lens)
    t, h_, d = int(cu[-1]), cfg.heads, cfg.head_dim
    x = np.empty((t, 3, h_, d), dtype=np.float32)
    for s in range(len(lens)):
        a, b = int(cu[s]), int(cu[s + 1])
        gs = s + seq_offset
        for h in range(h_):
            x[a:b, 0, h] = _rng(cfg.cfg_id, 0, gs, h, seed).standard_normal((b - a, d), dtype=np.float32)
            x[a:b, 1, h] = _rng(cfg.cfg_id, 1, gs, h, seed).standard_normal((b - a, d), dtype=np.float32)
            x[a:b, 2, h] = _rng(cfg.cfg_id, 2, gs, h, seed).uniform(-1.0, 1.0, (b - a, d)).astype(np.float32)
    return _round(x, cfg.torch_dtype), cu


def _round(x32: np.ndarray, tdtype) -> torch.Tensor:
    # torch's float32 -> fp16/bf16 conversion is round-to-nearest-even
    return torch.from_numpy(np.ascontiguousarray(x32, dtype=np.float32)).to(tdtype)


def _rng(cfg_id: int, tensor_id: int, b: int, h: int, seed: int = SEED):
    return np.random.default_rng(np.random.SeedSequence([seed, cfg_id, tensor_id, b, h]))


def kv_lengths(cfg: FmhaConfig, batch_offset: int = 0, seed: int = SEED) -> np.ndarray | None:
    """Per-batch valid key count for key-padding configs (right padding)."""
    if cfg.mask != MASK_KEY_PADDING:
        return None
    out = np.empty(cfg.batch, dtype=np.int32)
    for b in range(cfg.batch):
        gb = b + batch_offset
        if gb == 0:
            out[b] = cfg.seq_kv
        else:
            lo = min(32, cfg.seq_kv)
            out[b] = _rng(cfg.cfg_id, 9, gb, 0, seed).integers(lo, cfg.seq_kv + 1)
    return out


def make_fmha_inputs(cfg: FmhaConfig, batch_offset: int = 0, seed: int = SEED):
    """Returns (q, k, v, kv_len) as CPU torch tensors [B,H,S,D] in cfg's dtype
    (kv_len: int32 numpy array or None).  Global batch index = b + batch_offset."""
    b_, h_, sq, skv, d = cfg.batch, cfg.heads, cfg.seq_q, cfg.seq_kv, cfg.head_dim
    q = np.empty((b_, h_, sq, d), dtype=np.float32)
    k = np.empty((b_, h_, skv, d), dtype=np.float32)
    v = np.empty((b_, h_, skv, d), dtype=np.float32)
    for b in range(b_):
        gb = b + batch_offset
        for h in range(h_):
            q[b, h] = _rng(cfg.cfg_id, 0, gb, h, seed).standard_normal((sq, d), dtype=np.float32) * cfg.qk_sigma
            k[b, h] = _rng(cfg.cfg_id, 1, gb, h, seed).standard_normal((skv, d), dtype=np.float32) * cfg.qk_sigma
            v[b, h] = _rng(cfg.cfg_id, 2, gb, h, seed).uniform(-1.0, 1.0, (skv, d)).astype(np.float32)
    td = cfg.torch_dtype
    return _round(q, td), _round(k, td), _round(v, td), kv_lengths(cfg, batch_offset, seed)


def shard(cfg: FmhaConfig, rank: int, world: int, scaling: str = "weak"):
    """The multi-GPU partition: every (b, h) is independent, so ranks split by batch.
    weak:   every rank runs the whole config on its own batch (global batch = world * cfg.batch);
    strong: the config's batch is split into `world` contiguous ranges (batch must divide).
    Returns (local config, global batch offset)."""
    if scaling == "weak":
        return cfg, rank * cfg.batch
    if scaling != "strong":
        raise ValueError(scaling)
    if cfg.batch % world:
        raise ValueError(f"batch {cfg.batch} does not split over {world} ranks")
    b = cfg.batch // world
    return cfg.with_(batch=b), rank * b


def make_mlp_inputs(cfg: MlpConfig = MLP_CONFIG, tokens: int | None = None, seed: int = SEED):
    """Returns (x [T,d_model], w1 [d_ff,d_model], b1 [d_ff], w2 [d_model,d_ff], b2 [d_model])
    as fp16 CPU tensors."""
    t = cfg.tokens if tokens is None else tokens
    r = lambda tid: _rng(cfg.cfg_id, tid, 0, 0, seed)
    x = r(0).uniform(-1, 1, (t, cfg.d_model)).astype(np.float32)
    w1 = (r(1).standard_normal((cfg.d_ff, cfg.d_model), dtype=np.float32) / np.sqrt(cfg.d_model)).astype(np.float32)
    b1 = r(2).uniform(-1, 1, cfg.d_ff).astype(np.float32)
    w2 = (r(3).standard_normal((cfg.d_model, cfg.d_ff), dtype=np.float32) / np.sqrt(cfg.d_ff)).astype(np.float32)
    b2 = r(4).uniform(-1, 1, cfg.d_model).astype(np.float32)
    td = torch.float16
    return tuple(_round(a, td) for a in (x, w1, b1, w2, b2))


def make_gemm_inputs(m: int, n: int, k: int, seed: int = SEED, cfg_id: int = 7):
    """Generic GEMM+bias test inputs: A ~ U(-1,1) [M,K], W ~ N(0,1/K) [N,K], b ~ U(-1,1) [N]."""
    r = lambda tid: _rng(cfg_id, tid, m, n * 100003 + k, seed)
    a = r(0).uniform(-1, 1, (m, k)).astype(np.float32)
    w = (r(1).standard_normal((n, k), dtype=np.float32) / np.sqrt(max(k, 1))).astype(np.float32)
    b = r(2).uniform(-1, 1, n).astype(np.float32)
    td = torch.float16
    return _round(a, td), _round(w, td), _round(b, td)


@dataclass(frozen=True)
class LayerConfig:
    """Synthetic Transformer layer: packed tokens of num_seqs sequences."""
    name: str
    cfg_id: int
    num_seqs: int
    seq_len: int          # every sequence's length (equal lengths) unless lengths are passed
    d_model: int
    heads: int
    d_ff: int
    causal: bool = False

    @property
    def head_dim(self) -> int:
        return self.d_model // self.heads

    @property
    def scale(self) -> float:
        return float(np.float32(1.0 / np.sqrt(self.head_dim)))

    def with_(self, **kw) -> "LayerConfig":
        return replace(self, **kw)


# BERT-large layer at BASELINE.json config 5's token count: 32 sequences x 512 tokens = 16384 tokens,
# d_model 1024, 16 heads (D = 64), d_ff 4096 (BJ configs 3 and 5)
LAYER_CONFIGS = {
    "bert_layer": LayerConfig("bert_layer", 10, 32, 512, 1024, 16, 4096),
}


def make_layer_inputs(cfg: LayerConfig, lengths=None, seed: int = SEED):
    """Returns (x, wqkv, bqkv, wo, bo, w1, b1, w2, b2) fp16 CPU tensors and cu_seqlens (int32 numpy).
    x ~ U(-1, 1) [T, d]; every W ~ N(0, 1/fan_in) in nn.Linear layout [out, in]; biases ~ U(-1, 1)."""
    lens = np.full(cfg.num_seqs, cfg.seq_len, dtype=np.int64) if lengths is None else np.asarray(lengths)
    cu = np.zeros(len(lens) + 1, dtype=np.int32)
    cu[1:] = np.cumsum(lens)
    t, d, f = int(cu[-1]), cfg.d_model, cfg.d_ff
    r = lambda tid: _rng(cfg.cfg_id, tid, 0, 0, seed)
    w = lambda tid, o, i: (r(tid).standard_normal((o, i), dtype=np.float32) / np.sqrt(i)).astype(np.float32)
    b = lambda tid, o: r(tid).uniform(-1, 1, o).astype(np.float32)
    arrs = [r(0).uniform(-1, 1, (t, d)).astype(np.float32), w(1, 3 * d, d), b(2, 3 * d), w(3, d, d), b(4, d),
            w(5, f, d), b(6, f), w(7, d, f), b(8, d)]
    return tuple(_round(a, torch.float16) for a in arrs), cu

@dataclass(frozen=True)
class FusedMlpConfig:
    """The paper's fused multi-layer MLP (Fig. 11): `layers` chained GEMM + bias + ReLU
    layers of width N = K <= 128 over M rows.  The paper gives no M; 65536 rows is an assumption
    (DESIGN.md §4)."""
    name: str
    cfg_id: int
    m: int
    width: int
    layers: int


FUSED_MLP_CONFIGS = {
    "mlp_fused": FusedMlpConfig("mlp_fused", 12, 65536, 128, 20),
    "mlp_fused_w64": FusedMlpConfig("mlp_fused_w64", 13, 65536, 64, 20),
}


def make_fused_mlp_inputs(m: int, width: int, layers: int, seed: int = SEED, cfg_id: int = 12):
    """x ~ U(-1, 1) [M, N]; W_l ~ N(0, 2/N) [L, N, N] (He scaling, so activations keep their size
    through ReLU layers); b_l ~ U(-0.1, 0.1) [L, N].  fp16 CPU tensors (RNE from fp32)."""
    r = lambda tid: _rng(cfg_id, tid, m, width * 1000 + layers, seed)
    x = r(0).uniform(-1, 1, (m, width)).astype(np.float32)
    w = (r(1).standard_normal((layers, width, width), dtype=np.float32) * np.sqrt(2.0 / width)).astype(np.float32)
    b = r(2).uniform(-0.1, 0.1, (layers, width)).astype(np.float32)
    return tuple(_round(a, torch.float16) for a in (x, w, b))


# ------------------------------------------------------------------ score-ramp inputs (lazy rescale)
def ramp_spikes(seq_kv: int, tile: int = 128):
    """Positions of the 'spike' keys of the score-ramp inputs: one key per `tile`-key block t, at
    128 t + (7 + 37 t) % 128 (t = 0 has none).  Returns a list of (t, key index)."""
    return [(t, t * tile + (7 + 37 * t) % tile) for t in range(1, (seq_kv + tile - 1) // tile)
            if t * tile + (7 + 37 * t) % tile < seq_kv]


def add_score_ramp(q: torch.Tensor, k: torch.Tensor, scale: float, step_log2: float = 9.0):
    """Score-ramp variant of [.., S, D] inputs (q, k CPU tensors, modified copies returned): feature 0
    of every query row i gets a_i = (0, 0.5, 1, 2)[i % 4] and feature 0 of spike key t (see
    ramp_spikes) gets t * step_log2 * ln(2) / scale, so row i's largest score grows by about
    a_i * step_log2 (in log2 units) at every 128-key block: rows with a_i >= 1 move their max by
    more than 8 (log2) from one KV tile to the next, a_i = 0.5 every second tile, a_i = 0 never.
    Input construction only (no arithmetic of the method); feature 0 of the other keys is 0."""
    q, k = q.clone(), k.clone()
    sq, skv = q.shape[-2], k.shape[-2]
    a = torch.tensor([0.0, 0.5, 1.0, 2.0], dtype=torch.float32)[torch.arange(sq) % 4]
    q[..., :, 0] = a.to(q.dtype)
    k[..., :, 0] = 0
    for t, j in ramp_spikes(skv):
        k[..., j, 0] = float(t * step_log2 * np.log(2.0) / scale)
    return q, k
