"""Scheduling choices a plan learns from its previous checks (api.cpp choose_main_passes,
PgParams::seq_pref): a kernel whose optimistic pass flags at least half of
its instances runs its exact pass as the main pass, and a launch whose sequential re-run
found an XB race in at least half of its instances skips the block-parallel passes.  They
change which passes run, never the results: every repetition must equal the oracle bit for
bit."""
import pytest

from test_gpu_parity import assert_same, env, ir, run_pair  # noqa: F401  (env: fixture)

pytestmark = pytest.mark.gpu


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


def test_repeated_c1_takes_xb_launches_sequentially(env, oracle, W):
    """C1 (configs[0]): every non-square launch of the shared-memory transpose races between
    blocks (X4), so from the second check on its instances go straight to the sequential
    pass; the square ones stay block-parallel."""
    w = W.c1(n_seeds=8)
    ls = w.launch_src[::3]
    ref = oracle.check_parallel(W.subject(w.src), W.subject(w.tgt), ls, n_seeds=8, cap=1 << 20)
    pgvc, torch = env
    sp = pgvc.Space(ls, n_seeds=8, stream=torch.cuda.current_stream().cuda_stream)
    for _ in range(3):
        recs, summ = pgvc.check_equiv(ir(pgvc, W.subject(w.src)), ir(pgvc, W.subject(w.tgt)), sp).collect(cap=1 << 20)
        assert_same(ref, recs, summ)
    assert summ["per_kind"][4] > 0   # XB
