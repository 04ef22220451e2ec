"""GPU <-> oracle parity for the configuration-bug and bit-width sweeps (SURVEY.md §8(f)
NEXT-3): scalar product over ACCN = 1..16 in property mode and
the Table II transpose / reduction sweeps at 8/12/16/32-bit arithmetic (L895-L949)."""
import pytest

from test_gpu_parity import assert_same, run_pair
from test_gpu_property import env, run_prop  # noqa: F401  (fixture)

pytestmark = pytest.mark.gpu

FAILING = {0, 1, 2, 3, 4, 5, 9}


def test_accn_sweep(env, oracle, W):  # noqa: F811
    ls = W.accn_sweep(max_accn=16, bdims=(1, 4, 8), elementN=40)
    summ = run_prop(env, oracle, W, "scalar_prod", "post_scalar_prod", ls, n_seeds=4)
    assert summ["first_launch"] == 6            # ACCN = 3, bdim = 1 (launch order: ACCN-major)


@pytest.mark.parametrize("bits", [8, 16, 32])
def test_table2_transpose_bitwidths(env, oracle, W, bits):  # noqa: F811
    ls = []
    for n in (4, 8, 16, 32):
        for bx in range(1, n + 1):
            if n % bx == 0:
                ls.append(((1, 1, 1), (bx, n // bx, 1), (bx, n // bx)))
                ls.append(((2, 2, 1), (bx, n // bx, 1), (2 * bx, 2 * (n // bx))))
    ref, recs, summ, _ = run_pair(env, oracle, W.subject("naive_transpose"), W.subject("optimized_transpose"), ls,
                                  n_seeds=3, bits=bits)
    assert_same(ref, recs, summ)
    failed = {r[3] for r in recs if r[2] in FAILING}
    assert all((i in failed) == (l[1][0] != l[1][1]) for i, l in enumerate(ls))


@pytest.mark.parametrize("bits", [8, 12, 16, 32])
def test_table2_reduction_bitwidths(env, oracle, W, bits):  # noqa: F811
    for tgt in ("reduce1", "reduce2", "reduce3"):
        ls = [W.reduce_launch("reduce0", n, n) for n in (4, 8, 16, 32)]
        lt = [W.reduce_launch(tgt, n, n) for n in (4, 8, 16, 32)]
        ref, recs, summ, _ = run_pair(env, oracle, W.subject("reduce0"), W.subject(tgt), ls, lt, n_seeds=3, bits=bits)
        assert_same(ref, recs, summ)
