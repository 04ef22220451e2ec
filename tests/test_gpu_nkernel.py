"""GPU parity of the N-kernel comparative assertion (pg_check_equiv_n; SURVEY.md §8(d) C2
design): every kernel once per (launch, seed), all pairs compared,
bit-exact against oracle.check_n - record lists, counts, first keys."""
import pytest

from test_gpu_parity import assert_same, env, ir  # noqa: F401  (env: fixture)

pytestmark = pytest.mark.gpu


def _gpu(env, W, names, launches, n_seeds, checks=7, seed_base=0):
    pgvc, torch = env
    sp = pgvc.Space(launches[0], n_seeds=n_seeds, seed_base=seed_base, checks=checks,
                    stream=torch.cuda.current_stream().cuda_stream)
    run = pgvc.check_equiv_n([ir(pgvc, W.subject(n)) for n in names], launches, sp)
    return run.collect(cap=1 << 20)


@pytest.mark.parametrize("group", [0, 1])
def test_c2_all_reduced(env, oracle, W, group):
    w = W.c2_all(n_seeds=3, max_log_n=10, max_log_b=9)[group]
    ref = oracle.check_n_parallel([W.subject(n) for n in w.kernels], w.launches, n_seeds=3, cap=1 << 20)
    recs, summ = _gpu(env, W, w.kernels, w.launches, 3)
    assert_same(ref, recs, summ)


def test_mismatch_slots_and_sites(env, oracle, W):
    names = ["reduce0", "reduce1", "reduce2", "reduce0_lit", "reduce3"]
    pts = W.c2_points(9, 8, 1)
    lists = [[W.reduce_launch("reduce0" if n == "reduce0_lit" else n, N, B) for N, B in pts] for n in names]
    ref = oracle.check_n_parallel([W.subject(n) for n in names], lists, n_seeds=5, seed_base=11, cap=1 << 20)
    recs, summ = _gpu(env, W, names, lists, 5, seed_base=11)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][5] > 0 and {r[7] for r in recs if r[2] == 5} >= {3, 4}


@pytest.mark.timeout(2400)
@pytest.mark.parametrize("group", [0, 1])
def test_c2_all_bench_space_nine_seeds(env, oracle, W, group):
    w = W.c2_all(n_seeds=9)[group]                 # N <= 2^16, B <= 2^10: the bench's space
    ref = oracle.check_n_parallel([W.subject(n) for n in w.kernels], w.launches, n_seeds=9, cap=1 << 20)
    recs, summ = _gpu(env, W, w.kernels, w.launches, 9)
    assert_same(ref, recs, summ)

