"""Configuration bugs and bit-width sweeps on the oracle.

* Scalar product with ACCN not a power of two: the post-condition
  kernel is pinned to numpy's dot product; every power-of-two ACCN satisfies it, the
  first violation in ACCN order is ACCN = 3, and every non-power-of-two ACCN fails
  once elementN >= ACCN (the tree's first stride ACCN/2 drops partial sums).
* Table II (L895-L949) verdicts at 8/16/32-bit arithmetic: transposes are equivalent
  only for square blocks at every width; reduce0 and reduce1 agree at 8/12/16/32 bits."""
import os

import numpy as np

FAILING = {0, 1, 2, 3, 4, 5, 9}


def test_post_scalar_prod_closed_form(oracle, W):
    for vN, eN in [(1, 5), (3, 17), (2, 64)]:
        l = W.property_launches([W.scalar_prod_launch(vN, eN, 4, 4)], 6)[0]
        init, fin, _ = oracle.exec_kernel(W.subject("post_scalar_prod"), l, 9)
        a = init[0].astype(np.uint64).reshape(vN, eN)      # d_A, d_B, d_C (sorted names)
        b = init[1].astype(np.uint64).reshape(vN, eN)
        want = ((a * b) % (1 << 32)).sum(axis=1) % (1 << 32)
        assert (fin[2] == want.astype(np.uint32)).all()


def prop(oracle, W, ls, n_seeds=2):
    lt = W.property_launches(ls, 6)
    return oracle.check(W.subject("scalar_prod"), W.subject("post_scalar_prod"), ls, lt, n_seeds=n_seeds)


def test_accn_power_of_two_only(oracle, W):
    ls = W.accn_sweep(max_accn=16, bdims=(1, 4), elementN=40)
    r = prop(oracle, W, ls)
    failed = {x[3] for x in r["records"] if x[2] in FAILING}
    for i, l in enumerate(ls):
        accn = l.scalars[2]
        assert (i in failed) == (accn & (accn - 1) != 0), (accn, l.bdim)
    assert r["first_key"][0] >> 45 == 4          # first failing launch: ACCN = 3 (index 2*2)


def test_table2_bitwidths(oracle, W):
    golden = []
    with open(os.path.join(os.path.dirname(__file__), "golden", "table2_transpose_verdicts.txt")) as f:
        for line in f:
            if line.strip() and not line.startswith("#"):
                n, star = line.split()
                golden.append((int(n), int(star)))
    src, tgt = W.subject("naive_transpose"), W.subject("optimized_transpose")
    for bits in (8, 16, 32):
        for n, star in golden:
            shapes = [(bx, n // bx) for bx in range(1, n + 1) if n % bx == 0]
            ls = [((1, 1, 1), (bx, by, 1), (bx, by)) for bx, by in shapes]
            r = oracle.check(src, tgt, ls, ls, n_seeds=2, bits=bits)
            failed = {x[3] for x in r["records"] if x[2] in FAILING}
            eq = [shapes[i] for i in range(len(ls)) if i not in failed]
            assert bool(star) == (len(eq) == 0), (bits, n)
            assert all(bx == by for bx, by in eq)
    r0, r1 = W.subject("reduce0"), W.subject("reduce1")
    for bits in (8, 12, 16, 32):
        ls = [W.reduce_launch("reduce0", n, n) for n in (4, 8, 16, 32)]
        r = oracle.check(r0, r1, ls, ls, n_seeds=3, bits=bits)
        if bits > 8:
            assert r["counts"][12] == 0, bits
            continue
        # 8-bit arithmetic: reduce1's index 2*k*tid wraps to 0 at k = 8, tid = 16 (n = 32),
        # so threads 0 and 16 both write sdata[0]: a WW race the wider widths do not have
        assert r["counts"][12] == 3                       # the three seeds of n = 32
        first = dict(zip(oracle.REC_FIELDS, r["records"][0]))
        assert (first["launch"], first["kernel"], first["kind"], first["addr"], first["tid_a"], first["tid_b"]) == \
            (3, 1, 2, 0, 0, 16)
