"""GPU VC-literal mode:
a second data-flow path on the device.  For every read the kernel also enumerates, for every
earlier round, every thread s of that round and tests "s wrote the cell" on s's logged
writes - the instantiated p(s) ∧ a = e(s) - and compares that literal writer with the
owner-stamp writer the data-flow row (H5) records.  Zero disagreements are required, and the
rows themselves must equal the oracle's, which are cross-checked by the oracle's own,
independent VC-literal re-evaluation (test_oracle_vcliteral.py)."""
import pytest

from test_gpu_dataflow import check_dataflow, env  # noqa: F401  (fixture)

pytestmark = pytest.mark.gpu


def _literal(env, text, launches, n_seeds=2, seed_base=7):
    pgvc, torch = env
    sp = pgvc.Space(launches, n_seeds=n_seeds, seed_base=seed_base,
                    checks=pgvc.CHK_RACE | pgvc.CHK_OOB | pgvc.CHK_VCLITERAL,
                    stream=torch.cuda.current_stream().cuda_stream)
    run = pgvc.check_races(pgvc.load_ir(text), sp)
    v = run.vcliteral()
    rows = run.dataflow()
    return v, rows


CASES = [
    ("naive_transpose", lambda W: [W.Launch((2, 2, 1), (4, 4, 1), (8, 8)), W.Launch((3, 2, 1), (4, 2, 1), (10, 7))]),
    ("optimized_transpose", lambda W: [W.Launch((2, 2, 1), (4, 4, 1), (8, 8)), W.Launch((3, 2, 1), (4, 2, 1), (10, 7))]),
    ("reduce0", lambda W: [W.reduce_launch("reduce0", 64, 16), W.reduce_launch("reduce0", 64, 64)]),
    ("reduce1", lambda W: [W.reduce_launch("reduce1", 64, 16), W.reduce_launch("reduce1", 128, 64)]),
    ("reduce2_obo", lambda W: [W.reduce_launch("reduce2_obo", 64, 16), W.reduce_launch("reduce2_obo", 32, 32)]),
    ("reduce6", lambda W: [W.reduce_launch("reduce6", 256, 64), W.reduce_launch("reduce6", 128, 128)]),
    ("prescan_nobarrier", lambda W: [W.scan_launch("prescan_nobarrier", 32, 8), W.scan_launch("prescan_nobarrier", 64, 16)]),
    ("prescan_padded", lambda W: [W.scan_launch("prescan_padded", 64, 16)]),
    ("bitonic_global", lambda W: [W.bitonic_launch("bitonic_global", 16), W.bitonic_launch("bitonic_global", 32)]),
    ("matmul_tiled_nobarrier", lambda W: [W.Launch((2, 2, 1), (4, 4, 1), (8, 8, 8))]),
]


@pytest.mark.parametrize("name,ls", CASES, ids=[c[0] for c in CASES])
def test_literal_writer_equals_owner_stamps(env, oracle, W, name, ls):
    launches = ls(W)
    v, rows = _literal(env, W.subject(name), launches)
    assert v["checked"] > 0 and v["overflow"] == 0
    assert v["disagree"] == 0, v
    # the rows of the literal run are the data-flow relation itself: equal to the oracle's
    check_dataflow(env, oracle, W.subject(name), launches)


def test_literal_mode_limits(env, W):
    pgvc, torch = env
    with pytest.raises(pgvc.PgError) as e:
        _literal(env, W.subject("reduce0"), [W.reduce_launch("reduce0", 256, 128)])
    assert e.value.code == pgvc.PG_E_LIMIT                       # n <= 64 threads per block
    run = pgvc.check_races(pgvc.load_ir(W.subject("reduce1")),
                           pgvc.Space([W.reduce_launch("reduce1", 16, 8)],
                                      stream=torch.cuda.current_stream().cuda_stream))
    with pytest.raises(pgvc.PgError) as e:
        run.vcliteral()
    assert e.value.code == pgvc.PG_E_STATE
