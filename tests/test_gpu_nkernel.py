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


def test_repeated_check_switches_main_pass(env, oracle, W):
    """A plan whose optimistic pass flags at least half of a kernel's instances (the injected
    off-by-one races in every instance with B >= 2) runs that kernel's exact pass as its main
    pass from the next check on (api.cpp choose_main_passes; a scheduling choice, DESIGN.md
    §5.5).  Every repetition - optimistic pass + re-run, then exact main pass - must equal
    the oracle bit for bit."""
    w = W.c2_all(n_seeds=9, max_log_n=12, max_log_b=10)[0]
    assert "reduce2_obo" in w.kernels
    ref = oracle.check_n_parallel([W.subject(n) for n in w.kernels], w.launches, n_seeds=9, cap=1 << 20)
    pgvc, torch = env
    sp = pgvc.Space(w.launches[0], n_seeds=9, checks=7, stream=torch.cuda.current_stream().cuda_stream)
    irs = [ir(pgvc, W.subject(n)) for n in w.kernels]
    for _ in range(3):
        recs, summ = pgvc.check_equiv_n(irs, w.launches, sp).collect(cap=1 << 20)
        assert_same(ref, recs, summ)


def test_repeated_pair_check_switches_main_pass(env, oracle, W):
    w = W.c2_pair("reduce2", "reduce2_obo", n_seeds=9, max_log_n=11, max_log_b=10)
    ref = oracle.check_parallel(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=9,
                                cap=1 << 20)
    pgvc, torch = env
    sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=9, stream=torch.cuda.current_stream().cuda_stream)
    for _ in range(3):
        recs, summ = pgvc.check_equiv(ir(pgvc, W.subject(w.src)), ir(pgvc, W.subject(w.tgt)), sp).collect(cap=1 << 20)
        assert_same(ref, recs, summ)
