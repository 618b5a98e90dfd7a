"""The algebra the time-segmented walk kernels rest on,
checked by brute force on the CPU, independently of the oracle and of CUDA.

Every open-loop round applies to the level one of: hold, +step (Alg. 3 l.18,
f4: min(l + s, r_max)), -step (l.23-25: max(l - s, r_min)), override to max
(l.10).  The kernels represent any composition of these as the clamp-shift
map l -> min(max(l + d, a), b) with d saturated to +-(r_max - r_min), packed
into 8-bit fields, and compose a word's actions sparsely (everything up to
the last override collapses to the constant r_max).  Here both shortcuts
are replayed in Python exactly as written in kernels_walk.cu and compared
with applying the rounds one by one, for every carry-in level.
"""
from __future__ import annotations

import random

import pytest

HOLD, UP, DOWN, OVR = 0, 1, 2, 3


def apply_round(l, act, step, lmin, lmax):
    if act == OVR:
        return lmax
    if act == UP:
        return min(l + step, lmax)
    if act == DOWN:
        return max(l - step, lmin)
    return l


def compose_dense(acts, step, lmin, lmax):
    """walk_map_kernel before the sparse rewrite: one map update per round."""
    K = lmax - lmin
    d, lo, hi = 0, lmin, lmax
    for act in acts:
        if act == OVR:
            d, lo, hi = 0, lmax, lmax
            continue
        sd = step if act == UP else (-step if act == DOWN else 0)
        d = min(max(d + sd, -K), K)
        lo = min(max(lo + sd, lmin), lmax)
        hi = min(max(hi + sd, lmin), lmax)
    return d, lo, hi


def compose_sparse_word(m, inc, dcr, hw, step, lmin, lmax):
    """The per-word composition of walk_map_kernel: collapse at the last
    override, then visit the remaining +-step bits in ascending order."""
    K = lmax - lmin
    d, lo, hi = m
    acts = inc | dcr
    if hw:
        j = hw.bit_length() - 1
        d, lo, hi = 0, lmax, lmax
        acts = 0 if j == 31 else acts & ((0xFFFFFFFE << j) & 0xFFFFFFFF)
    while acts:
        i = (acts & -acts).bit_length() - 1
        acts &= acts - 1
        sd = step if (inc >> i) & 1 else -step
        d = min(max(d + sd, -K), K)
        lo = min(max(lo + sd, lmin), lmax)
        hi = min(max(hi + sd, lmin), lmax)
    return d, lo, hi


def pack(d, a, b):
    return (d & 0xFF) | (a << 8) | (b << 16)


def apply_packed(m, l):
    d = m & 0xFF
    d = d - 256 if d >= 128 else d
    a, b = (m >> 8) & 0xFF, (m >> 16) & 0xFF
    return min(max(l + d, a), b)


def random_word(rng, p_act, p_ovr):
    """Masks as pass 1 writes them: +1 and -1 exclusive; hi independent
    (an override happens whatever Alg. 1 says)."""
    inc = dcr = hw = 0
    for i in range(32):
        if rng.random() < p_ovr:
            hw |= 1 << i
        r = rng.random()
        if r < p_act / 2:
            inc |= 1 << i
        elif r < p_act:
            dcr |= 1 << i
    return inc, dcr, hw


def word_acts(inc, dcr, hw):
    out = []
    for i in range(32):
        if (hw >> i) & 1:
            out.append(OVR)
        elif (inc >> i) & 1:
            out.append(UP)
        elif (dcr >> i) & 1:
            out.append(DOWN)
        else:
            out.append(HOLD)
    return out


@pytest.mark.parametrize("lmin,lmax", [(8, 22), (8, 25), (1, 127), (5, 6)])
def test_dense_composition_equals_sequential(lmin, lmax):
    rng = random.Random(lmin * 1000 + lmax)
    for trial in range(400):
        step = rng.choice([1, 2, 3, lmax - lmin, lmax - lmin + 5])
        n = rng.randint(0, 300)
        acts = [rng.choices([HOLD, UP, DOWN, OVR], weights=[5, 3, 3, 1 if trial % 3 else 0])[0] for _ in range(n)]
        m = pack(*compose_dense(acts, step, lmin, lmax))
        for carry in range(lmin, lmax + 1):
            l = carry
            for act in acts:
                l = apply_round(l, act, step, lmin, lmax)
            assert apply_packed(m, carry) == l, (trial, carry)


@pytest.mark.parametrize("lmin,lmax", [(8, 22), (1, 127), (10, 11)])
def test_sparse_word_composition_equals_sequential(lmin, lmax):
    rng = random.Random(7 + lmin)
    for trial in range(300):
        step = rng.choice([1, 2, 4, lmax - lmin])
        words = [random_word(rng, rng.choice([0.0, 0.2, 0.9]), rng.choice([0.0, 0.02, 0.3]))
                 for _ in range(rng.randint(1, 12))]
        m = (0, lmin, lmax)
        for inc, dcr, hw in words:
            m = compose_sparse_word(m, inc, dcr, hw, step, lmin, lmax)
        packed = pack(*m)
        for carry in range(lmin, lmax + 1):
            l = carry
            for inc, dcr, hw in words:
                for act in word_acts(inc, dcr, hw):
                    l = apply_round(l, act, step, lmin, lmax)
            assert apply_packed(packed, carry) == l, (trial, carry)


def test_segment_maps_chain_to_the_carry():
    """Carry-in of segment s = maps 0..s-1 applied to r_max in order (the
    prologue of walk_replay_kernel) equals the one-pass walk at t0 - 1."""
    rng = random.Random(3)
    lmin, lmax, step = 8, 22, 2
    acts = [rng.choices([HOLD, UP, DOWN, OVR], weights=[8, 3, 3, 1])[0] for _ in range(32 * 40)]
    seg = 96
    segs = [acts[i:i + seg] for i in range(0, len(acts), seg)]
    maps = [pack(*compose_dense(sg, step, lmin, lmax)) for sg in segs]
    l_true = lmax
    for s, sg in enumerate(segs):
        l = lmax
        for m in maps[:s]:
            l = apply_packed(m, l)
        assert l == l_true, s
        for act in sg:
            l_true = apply_round(l_true, act, step, lmin, lmax)
