"""Multi-seed lanes: the optimistic pass of a seed-oblivious kernel
carries PG_MS = 8 seeds per lane (PGVC_MS).  Seed counts that are not multiples of 8 leave
ragged seed groups; races, OOB and uninitialised reads inside a group flag all its
instances for the exact re-run, which runs the same seed groups (multi-seed exact
protocol).  Every case must equal the oracle bit for bit."""
import pytest

from test_gpu_parity import assert_same, env, run_pair  # noqa: F401  (fixture re-export)

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("pair,seeds", [(("reduce0", "reduce3"), 7), (("reduce2", "reduce2_obo"), 5),
                                        (("reduce0", "reduce6"), 9)])
def test_c2_ragged_seed_groups(env, oracle, W, pair, seeds):
    w = W.c2_pair(*pair, n_seeds=seeds, max_log_n=9, max_log_b=9)
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt,
                                  n_seeds=seeds, seed_base=31)
    assert_same(ref, recs, summ)


def test_c2_sharded_seed_groups(env, oracle, W):
    w = W.c2_pair("reduce0", "reduce4", n_seeds=10, max_log_n=8, max_log_b=8)
    for r in range(3):
        ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt,
                                      n_seeds=10, rank=r, world=3)
        assert_same(ref, recs, summ)


def test_c3_dropped_barrier_in_groups(env, oracle, W):
    w = W.c3_pair("prescan_nobarrier", 4, n_seeds=5, max_log_n=9, max_log_b=8)
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt,
                                  n_seeds=5)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][2] + summ["per_kind"][3] > 0   # the dropped barrier races


def test_c1_oob_in_groups(env, oracle, W):
    w = W.c1(n_seeds=6)
    ls = w.launch_src[:120]
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), ls, n_seeds=6, seed_base=5)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][1] > 0   # non-square blocks with bdim.y > bdim.x go out of bounds


def test_c5_matmul_trailing_barrier_in_groups(env, oracle, W):
    w = W.c5_matmul(n_seeds=3, sizes=(32, 64), K=64)
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject("matmul_tiled_nobarrier"), w.launch_src,
                                  n_seeds=3)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][3] > 0   # RW race, outputs still equal
