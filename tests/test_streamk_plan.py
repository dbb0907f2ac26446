"""Host logic of the stream-K tail (fmha_streamk_plan, fmha_streamk_workspace_bytes): no GPU needed.

The plan cuts each item of the persistent schedule's last, partial round into s key ranges of whole
128-key tiles; the pieces must still fit one round (rest * s <= SMs), every piece must hold at least
one key tile, s <= 4 (the kernel's merge registers), and the full rounds stay whole items."""

import math

import numpy as np
import pytest

import paper_conf_asplos_hagedornfccgg23_b200 as fm
from paper_conf_asplos_hagedornfccgg23_b200 import _lib

MASK_NONE, MASK_KEY_PADDING, MASK_CAUSAL, MASK_KEY_BIAS, MASK_ATTN_BIAS = 0, 1, 2, 3, 4


def pairs_across_units(b, h, nq, mask, sms):
    """fmha_fwd's pair_mode 1: odd q-tile counts >= 3, or 1 with more units than SMs."""
    return mask != MASK_CAUSAL and nq % 2 == 1 and (nq >= 3 or (nq == 1 and b * h > sms))


def singles(b, h, sq, items, mask, sms):
    nq = math.ceil(sq / 128)
    pair = pairs_across_units(b, h, nq, mask, sms)
    full = items // sms * sms
    rest_tiles = b * h * nq - 2 * full
    return pair and full > 0 and 0 < rest_tiles <= sms


def items_of(b, h, sq, mask, sms):
    """fmha_fwd's two-tile items: cross-unit pairs in pair_mode 1, else per-unit pairs."""
    nq = math.ceil(sq / 128)
    if pairs_across_units(b, h, nq, mask, sms):
        return (b * h * nq + 1) // 2
    return b * h * ((nq + 1) // 2)


def test_bert_large_384_on_148_sms():
    # 32 x 16 units x 3 q-tiles = 1536 tiles = 768 cross-unit pairs = 5 rounds of 148 + 28 (run as 56
    # single tiles by fmha_fwd); three key pieces would save less than the merge costs
    assert fm.streamk_plan(32, 16, 384, 384, 148) == (1, 0)
    assert fm.streamk_plan(8, 14, 384, 1024, 148) == (1, 0)  # (measured slower split)


def test_long_keys_split():
    # 3 x 50 units x 2 q-tile pairs... = 300 items = 2 rounds + 4; 32 KV tiles -> 4 pieces of 8
    assert fm.streamk_plan(3, 50, 512, 4096, 148) == (4, 4)


def test_bert_large_512_is_not_split():
    # 1024 items = 6 rounds + 136: 136 x 2 pieces would not fit one round
    assert fm.streamk_plan(32, 16, 512, 512, 148) == (1, 0)


def test_bias_masks_are_not_split():
    assert fm.streamk_plan(1, 3, 384, 384, 148, MASK_KEY_BIAS) == (1, 0)
    assert fm.streamk_plan(1, 3, 384, 384, 148, MASK_ATTN_BIAS) == (1, 0)


def test_single_key_tile_is_not_split():
    assert fm.streamk_plan(1, 3, 384, 128, 148) == (1, 0)


@pytest.mark.parametrize("seed", range(4))
def test_plan_invariants(seed):
    rng = np.random.default_rng(seed)
    for _ in range(400):
        b, h = int(rng.integers(1, 40)), int(rng.integers(1, 33))
        sq, skv = int(rng.integers(1, 3000)), int(rng.integers(1, 5000))
        mask = int(rng.choice([MASK_NONE, MASK_KEY_PADDING, MASK_CAUSAL]))
        sms = int(rng.choice([8, 132, 148]))
        s, tail = fm.streamk_plan(b, h, sq, skv, sms, mask)
        items = items_of(b, h, sq, mask, sms)
        nkv = math.ceil(skv / 128)
        if s == 1:
            assert tail == 0
            continue
        assert 2 <= s <= 4 and s <= nkv
        assert tail == items % sms and tail > 0
        assert tail * s <= sms                      # the pieces fit one round
        per = math.ceil(nkv / s)
        assert (s - 1) * per < nkv                  # every piece holds >= 1 key tile
        assert math.ceil(nkv / per) == s
        # the modelled last round (KV steps; fmha_fwd's singles ~0.65 of a pair step; merge ~2.5 steps)
        cost_fwd = (0.65 if singles(b, h, sq, items, mask, sms) else 1.0) * nkv
        assert cost_fwd - (per + 2.5) >= 1.5 - 1e-9


def test_workspace_bytes():
    lib = _lib.load()
    for d in (64, 128):
        got = lib.fmha_streamk_workspace_bytes(d, 148)
        # 148 counters (padded to 256 B) + 148 pieces x 2 tiles x 128 rows x (D + 2) floats
        assert got == 768 + 148 * 2 * 128 * (d + 2) * 4
    assert lib.fmha_streamk_workspace_bytes(96, 148) == 0
