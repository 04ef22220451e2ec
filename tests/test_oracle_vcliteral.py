"""P7: the data-flow relation computed from the ownership table equals the literal
instantiation of the paper's VCs: for every read,
enumerate every thread s of every earlier round and test "p(s) /\\ a = e(s)" (s wrote the
cell); the unique (or min-tid, under WW) such s of the latest such round is the writer."""
import pytest

CASES = [
    ("naive_transpose", "optimized_transpose", [((2, 2, 1), (2, 2, 1), (4, 4)), ((1, 2, 1), (3, 2, 1), (3, 4)),
                                                ((2, 1, 1), (2, 3, 1), (4, 3))]),
    ("reduce0", "reduce1", [((4, 1, 1), (8, 1, 1), (32,)), ((1, 1, 1), (6, 1, 1), (6,))]),
    ("reduce2", "reduce2_obo", [((2, 1, 1), (8, 1, 1), (16,))]),
    ("prescan", "prescan_nobarrier", [((2, 1, 1), (4, 1, 1), (16,))]),
    ("bitonic_global", None, [((1, 1, 1), (16, 1, 1), (16,))]),
    ("matmul_tiled", "matmul_tiled_nobarrier", [((2, 2, 1), (2, 2, 1), (4, 4, 4))]),
]


@pytest.mark.parametrize("src,tgt,launches", CASES)
def test_vc_literal_equals_ownership(oracle, W, src, tgt, launches):
    ts = W.subject(src)
    tt = W.subject(tgt) if tgt else None
    r = oracle.check(ts, tt, launches, launches if tt else None, n_seeds=3, vcliteral=True,
                     mode=0 if tt else 1)
    assert r["counts"][0] > 0
    for l in launches:
        rows = oracle.dataflow(ts, l, 1)
        assert len(rows) > 0
