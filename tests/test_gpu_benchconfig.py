"""Parity at the configuration bench.py times (BASELINE.json configs[1], C2): all seven
pairs - reduce0 against reduce1..6 and reduce2 against the injected off-by-one - over the
whole launch list (B = 2^0..2^10, N = B..2^16, so every B at N = 2^16), with nine seeds of
the bench's seed range: one full multi-seed group of PG_MS = 8 and a ragged group of one, so
the multi-seed optimistic pass and the multi-seed exact re-run of reduce2_obo run with full
groups exactly as in the timed step.  Plus C3 at n = 2^14 and C5 transpose at N = 1024 with
nine seeds.  Bit-exact against the oracle (run over the host cores, seed shards merged as
H9 merges ranks)."""
import pytest

from test_gpu_parity import assert_same, env, ir  # noqa: F401  (env: fixture)

pytestmark = pytest.mark.gpu


def _gpu(env, W, w, n_seeds, checks):
    pgvc, torch = env
    sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=n_seeds, checks=checks,
                    stream=torch.cuda.current_stream().cuda_stream)
    run = pgvc.check_equiv(ir(pgvc, W.subject(w.src)), ir(pgvc, W.subject(w.tgt)), sp)
    return run.collect(cap=1 << 20)


@pytest.mark.timeout(1800)
@pytest.mark.parametrize("pair", [("reduce0", "reduce1"), ("reduce0", "reduce2"), ("reduce0", "reduce3"),
                                  ("reduce0", "reduce4"), ("reduce0", "reduce5"), ("reduce0", "reduce6"),
                                  ("reduce2", "reduce2_obo")])
def test_c2_bench_space_nine_seeds(env, oracle, W, pair):
    w = W.c2_pair(*pair, n_seeds=9)            # the bench's launch list (N <= 2^16, B <= 2^10)
    assert max(l.scalars[0] for l in w.launch_src) == 1 << 16
    ref = oracle.check_parallel(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=9,
                                checks=w.checks, cap=1 << 20)
    recs, summ = _gpu(env, W, w, 9, w.checks)
    assert_same(ref, recs, summ)
    if pair[1] == "reduce2_obo":
        assert summ["n_fail"] > 0


@pytest.mark.timeout(1800)
@pytest.mark.parametrize("tgt,lognb", [("prescan_padded", 4), ("prescan_nobarrier", 4)])
def test_c3_full_size_nine_seeds(env, oracle, W, tgt, lognb):
    w = W.c3_pair(tgt, lognb, n_seeds=9, max_log_n=14)
    ls = [l for l in w.launch_src if l.scalars[0] == 1 << 14]       # every B at n = 2^14
    lt = [w.launch_tgt[i] for i, l in enumerate(w.launch_src) if l.scalars[0] == 1 << 14]
    ref = oracle.check_parallel(W.subject(w.src), W.subject(w.tgt), ls, lt, n_seeds=9, checks=w.checks,
                                cap=1 << 20)
    pgvc, torch = env
    sp = pgvc.Space(ls, lt, n_seeds=9, checks=w.checks, stream=torch.cuda.current_stream().cuda_stream)
    recs, summ = pgvc.check_equiv(ir(pgvc, W.subject(w.src)), ir(pgvc, W.subject(w.tgt)), sp).collect(cap=1 << 20)
    assert_same(ref, recs, summ)


@pytest.mark.timeout(1800)
def test_c5_transpose_1024_nine_seeds(env, oracle, W):
    w = W.c5_transpose(n_seeds=9, sizes=(1024,))
    ref = oracle.check_parallel(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=9,
                                checks=w.checks, cap=1 << 20)
    recs, summ = _gpu(env, W, w, 9, w.checks)
    assert_same(ref, recs, summ)
