"""Oracle pins for the bitonic pair."""
import numpy as np
import pytest


def sorted_signed(x):
    return np.sort(x.astype(np.int32)).astype(np.uint32)


@pytest.mark.parametrize("name", ["bitonic_global", "bitonic_shared"])
def test_sorts_random_and_tied_inputs(oracle, W, name):
    for n in (2, 4, 16, 128, 1024):
        l = W.bitonic_launch(name, n)
        for mode, rng in ((0, 0), (2, 4)):
            for seed in (1, 2):
                init, fin, counts = oracle.exec_kernel(W.subject(name), l, seed, input_mode=mode, input_range=rng)
                assert (fin[0] == sorted_signed(init[0])).all()
                assert sum(counts[1:11]) == 0


@pytest.mark.parametrize("n", [2, 4, 8])
def test_zero_one_principle_exhaustive(oracle, W, n):
    # 0-1 principle (Knuth): a comparator network sorts all inputs iff it sorts all 2^n 0/1 inputs.
    # BITS01 seed s gives a[i] = (s >> i) & 1, so seeds 0..2^n-1 enumerate every 0/1 input.
    src, tgt = W.subject("bitonic_global"), W.subject("bitonic_shared")
    ls, lt = [W.bitonic_launch("bitonic_global", n)], [W.bitonic_launch("bitonic_shared", n)]
    r = oracle.check(src, tgt, ls, lt, n_seeds=1 << n, input_mode=1)
    assert r["n_records"] == 0
    for s in (0, (1 << n) - 1, 0b0110 & ((1 << n) - 1)):
        init, fin, _ = oracle.exec_kernel(src, ls[0], s, input_mode=1)
        assert list(init[0]) == [(s >> i) & 1 for i in range(n)]
        assert list(fin[0]) == sorted(init[0])


@pytest.mark.slow
def test_zero_one_principle_n16(oracle, W):
    src, tgt = W.subject("bitonic_global"), W.subject("bitonic_shared")
    r = oracle.check(src, tgt, [W.bitonic_launch("bitonic_global", 16)], [W.bitonic_launch("bitonic_shared", 16)],
                     n_seeds=1 << 16, input_mode=1)
    assert r["n_records"] == 0


def test_round_counts_at_4096(oracle, W):
    # L = log2 n = 12: L(L+1)/2 = 78 compare-exchange rounds in both formulations; the global
    # version has 78 barriers (79 rounds), the shared one adds a load and a store round (80)
    n = 4096
    _, _, cg = oracle.exec_kernel(W.subject("bitonic_global"), W.bitonic_launch("bitonic_global", n), 1)
    _, _, cs = oracle.exec_kernel(W.subject("bitonic_shared"), W.bitonic_launch("bitonic_shared", n), 1)
    assert cg[0] == n * 79 and cs[0] == (n // 2) * 80
    assert sum(cg[1:11]) == 0 and sum(cs[1:11]) == 0
