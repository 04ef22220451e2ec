"""Pins for the N-kernel comparative assertion (SURVEY.md §8(d) C2 design: reduce0..6
pairwise, each kernel run once per instance; PAPER.md L820-L846 reduction-loop pairs).

What fixes the expected values: every correct SDK variant computes odata[b] = Σ of its
block's B inputs mod 2^32 (X11, L465), so all 21 pairs of reduce0..6 agree on every
instance; the injected off-by-one (L962-L964) differs from all of them exactly where the
two-kernel check says it differs from reduce2, and first at (N, B) = (2, 2)."""
import itertools

import pytest


def _sub(W, name):
    return W.subject(name)


def test_all_correct_variants_agree_pairwise(oracle, W):
    ws = W.c2_all(n_seeds=2, max_log_n=6, max_log_b=5)
    w = ws[0]
    k = w.kernels.index("reduce2_obo")
    texts = [_sub(W, n) for i, n in enumerate(w.kernels) if i != k]
    lists = [l for i, l in enumerate(w.launches) if i != k]
    r = oracle.check_n(texts, lists, n_seeds=2, cap=1 << 20)
    assert r["counts"][1 + 5] == 0 and r["first_key"][0] == 2 ** 63 - 1      # no MISMATCH, no failure
    # instances = the sum over kernels of each kernel's own race-mode run (each runs once)
    want = sum(oracle.check(t, None, l, mode=1, n_seeds=2)["counts"][0] for t, l in zip(texts, lists))
    assert r["counts"][0] == want


def test_mismatch_records_match_the_pair_checks(oracle, W):
    # reduce0_lit is the literal L825 header (X10): a wrong sum first at bdim = 4 (P3 (v)).  In
    # the 4-kernel check its mismatches land in the slots of kernels 0..2 with site = 3, and
    # each slot holds exactly the two-kernel check (i, reduce0_lit)'s MISMATCH record.
    names = ["reduce0", "reduce1", "reduce2", "reduce0_lit"]
    pts = W.c2_points(5, 4, 1)
    lists = [[W.reduce_launch("reduce0" if n == "reduce0_lit" else n, N, B) for N, B in pts] for n in names]
    texts = [_sub(W, n) for n in names]
    r = oracle.check_n(texts, lists, n_seeds=3, cap=1 << 20)
    mm = [x for x in r["records"] if x[2] == 5]
    assert mm and all(x[7] == 3 and x[5] < 3 for x in mm)
    for i in range(3):
        pair = oracle.check(texts[i], texts[3], lists[i], lists[3], n_seeds=3, cap=1 << 20)
        want = [x for x in pair["records"] if x[2] == 5]
        got = [x for x in mm if x[5] == i]
        assert len(got) == len(want) > 0
        for g, p in zip(got, want):
            assert g[1:5] == p[1:5] and g[6:7] == p[6:7] and g[8:] == p[8:]    # all but key / kernel / site
            assert p[7] == 0xFFFFFFFF
    first_b4 = min(i for i, (N, B) in enumerate(pts) if B == 4)
    assert r["first_key"][1 + 5] >> 45 == first_b4              # first MISMATCH at bdim = 4


def test_obo_fails_by_races_not_outputs(oracle, W):
    # the injected off-by-one (tid <= s) races and reads out of bounds but still sums
    # correctly under X3 (P3 (iv)): in the 8-kernel check it adds OOB / RW records of kernel 7
    # only, no MISMATCH
    w = W.c2_all(n_seeds=2, max_log_n=5, max_log_b=4)[0]
    r = oracle.check_n([_sub(W, n) for n in w.kernels], w.launches, n_seeds=2, cap=1 << 20)
    assert r["counts"][1 + 5] == 0
    ob = w.kernels.index("reduce2_obo")
    kinds = {(x[5], x[2]) for x in r["records"]}
    assert {k for k, _ in kinds} == {ob} and {1, 3} <= {kd for _, kd in kinds}
    assert r["first_key"][0] >> 45 == 0                          # (N, B) = (2, 2) fails at once


def test_b1_group_and_key_layout(oracle, W):
    w = W.c2_all(n_seeds=2, max_log_n=4, max_log_b=2)[1]
    assert w.kernels == ["reduce0", "reduce1", "reduce2", "reduce2_obo"]
    r = oracle.check_n([_sub(W, n) for n in w.kernels], w.launches, n_seeds=2, cap=1 << 20)
    for x in r["records"]:
        key, kind, launch, seed, kernel = x[0], x[2], x[3], x[4], x[5]
        # X16: launch (19) | seed_idx (21) | kernel (4) | kind (4) | round (16)
        assert key >> 45 == launch and (key >> 24) & 0x1FFFFF == seed and (key >> 20) & 0xF == kernel
        assert (key >> 16) & 0xF == kind
