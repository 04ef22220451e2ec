"""Minimal failing-n search (paper_conf_ipps_lig12_b200/search.py).

The search logic is host orchestration; here it drives the oracle (CPU) and the C ABI
(GPU) and must find the first witnesses the paper fixes: n = 2, bdim (2,1) for the
transpose pair (P2); (N, B) = (2, 2) for reduce2_obo (P3 iv); ACCN = 3 for the scalar
product (L956-L961) - while checking fewer launches than the whole space."""
import pytest

from paper_conf_ipps_lig12_b200 import search


def oracle_runner(oracle, W, src, tgt, tgt_of=None, n_seeds=2, post_scalars=None):
    def run(launches, offset):
        if post_scalars:
            lt = W.property_launches(launches, post_scalars)
        else:
            lt = [tgt_of(l) for l in launches] if tgt_of else launches
        r = oracle.check(W.subject(src), W.subject(tgt), list(launches), lt, n_seeds=n_seeds)
        k = r["first_key"][0]
        first = 0xFFFFFFFF if k == (1 << 63) - 1 else k >> 45
        return r["records"], {"first_launch": first}
    return run


def transpose_groups(W):
    groups = {}
    for l in W.c1_launches():
        groups.setdefault(l.threads, []).append(l)
    return sorted(groups.items())


def test_search_transpose_first_witness(oracle, W):
    groups = transpose_groups(W)
    w = search.first_failing(groups, oracle_runner(oracle, W, "naive_transpose", "optimized_transpose"))
    assert w.n == 2 and w.launch.bdim[:2] == (2, 1) and w.launch.gdim[:2] == (1, 1)
    assert w.launches_checked < sum(len(ls) for _, ls in groups)


def test_search_obo_and_no_failure(oracle, W):
    groups = [(B, [W.reduce_launch("reduce2", N, B) for N in (B, 4 * B)]) for B in (1, 2, 4, 8, 16)]
    w = search.first_failing(groups, oracle_runner(oracle, W, "reduce2", "reduce2_obo"))
    assert w.n == 2 and w.launch.scalars == (2,) and w.launch.bdim[0] == 2
    assert search.first_failing(groups, oracle_runner(oracle, W, "reduce0", "reduce1")) is None


def test_search_accn(oracle, W):
    groups = [(a, [W.scalar_prod_launch(2, 40, a, b) for b in (1, 4)]) for a in range(1, 17)]
    w = search.first_failing(groups, oracle_runner(oracle, W, "scalar_prod", "post_scalar_prod", post_scalars=6))
    assert w.n == 3 and w.calls == 2 and w.launches_checked == 6


@pytest.mark.gpu
def test_search_on_gpu(W):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_lig12_b200 import pgvc
    groups = transpose_groups(W)
    s, t = pgvc.load_ir(W.subject("naive_transpose")), pgvc.load_ir(W.subject("optimized_transpose"))
    w = search.first_failing(groups, search.equiv_runner(pgvc, s, t, n_seeds=4))
    assert w.n == 2 and w.launch.bdim[:2] == (2, 1)
    groups = [(a, [W.scalar_prod_launch(2, 40, a, b) for b in (1, 4, 8)]) for a in range(1, 17)]
    k, post = pgvc.load_ir(W.subject("scalar_prod")), pgvc.load_ir(W.subject("post_scalar_prod"))
    w = search.first_failing(groups, search.property_runner(pgvc, k, post, n_seeds=4))
    assert w.n == 3 and all(r[2] == 5 for r in w.records)      # MISMATCH records of that launch
