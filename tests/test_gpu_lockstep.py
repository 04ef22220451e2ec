"""GPU <-> oracle parity of the lock-step comparison (PG_CHK_LOCKSTEP, pg_collect_lockstep;
SURVEY.md §8(f) NEXT-2, X25): the first shared-state divergence of every
instance, row for row, on the aligned reduction loops, the scan
barrier mutant and the tiled-matmul barrier mutant."""
import pytest

from test_gpu_parity import env  # noqa: F401  (fixture)

pytestmark = pytest.mark.gpu


def both(env, oracle, W, src, tgt, ls, lt, n_seeds=3, **kw):  # noqa: F811
    pgvc, torch = env
    ref = oracle.lockstep(W.subject(src), W.subject(tgt), ls, lt, n_seeds=n_seeds, lock_rounds=32, **kw)
    sp = pgvc.Space(ls, lt, n_seeds=n_seeds, checks=pgvc.CHK_EQUIV | pgvc.CHK_RACE | pgvc.CHK_OOB | pgvc.CHK_LOCKSTEP,
                    stream=torch.cuda.current_stream().cuda_stream, **kw)
    run = pgvc.check_equiv(pgvc.load_ir(W.subject(src)), pgvc.load_ir(W.subject(tgt)), sp)
    got = run.lockstep()
    recs, summ = run.collect()
    assert got == ref
    return got, summ


@pytest.mark.parametrize("tgt", ["reduce1", "reduce2", "reduce2_obo", "reduce0_lit", "reduce3"])
def test_lockstep_reductions(env, oracle, W, tgt):  # noqa: F811
    pts = [(B, B) for B in (1, 2, 4, 8, 32, 64, 256)] + [(1024, 64), (4096, 1024)]
    if tgt in W.REDUCE_HALF:
        pts = pts[1:]                          # B/2-thread variants need B >= 2
    ls = [W.reduce_launch("reduce0", N, B) for N, B in pts]
    lt = [W.reduce_launch(tgt, N, B) for N, B in pts]
    rows, _ = both(env, oracle, W, "reduce0", tgt, ls, lt)
    if tgt == "reduce1":
        assert rows == []                      # identical shared state after every round (L839-L845)
    if tgt == "reduce3":
        assert rows == []                      # half-size blocks: sdata sizes differ, nothing compared


def test_lockstep_scan_and_matmul(env, oracle, W):  # noqa: F811
    ls = [W.scan_launch("prescan", n, B) for (n, B) in [(4, 2), (32, 4), (256, 32)]]
    lt = [W.scan_launch("prescan_nobarrier", n, B) for (n, B) in [(4, 2), (32, 4), (256, 32)]]
    rows, _ = both(env, oracle, W, "prescan", "prescan_nobarrier", ls, lt)
    assert rows
    ls = [((2, 2, 1), (4, 4, 1), (K, 8, 8)) for K in (4, 8, 12)]
    both(env, oracle, W, "matmul_tiled", "matmul_tiled_nobarrier", ls, ls, n_seeds=2)
