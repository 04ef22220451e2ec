"""Edge cases and limits of the C ABI on the GPU (include/pgvc.h conventions): empty
spaces, degenerate launches, argument and limit errors, record-buffer truncation,
the largest emulated block, and repeated / interleaved checks reusing cached plans."""
import pytest

from test_gpu_parity import assert_same, env, run_pair  # noqa: F401  (env: fixture)

pytestmark = pytest.mark.gpu


def _irs(pgvc, W, a, b):
    return pgvc.load_ir(W.subject(a)), pgvc.load_ir(W.subject(b))


def test_zero_seeds_is_an_empty_run(env, W):  # noqa: F811
    pgvc, torch = env
    s, t = _irs(pgvc, W, "reduce0", "reduce1")
    run = pgvc.check_equiv(s, t, pgvc.Space([W.reduce_launch("reduce0", 8, 4)], n_seeds=0))
    recs, summ = run.collect()
    assert recs == [] and summ["instances"] == 0 and summ["n_fail"] == 0 and summ["first_launch"] == 0xFFFFFFFF


def test_rank_beyond_seeds_is_empty(env, W):  # noqa: F811
    pgvc, torch = env
    s, t = _irs(pgvc, W, "reduce0", "reduce1")
    run = pgvc.check_equiv(s, t, pgvc.Space([W.reduce_launch("reduce0", 8, 4)], n_seeds=2, rank=3, world=4))
    recs, summ = run.collect()
    assert summ["instances"] == 0


@pytest.mark.parametrize("space, code", [
    (dict(launch_src=[]), "ARG"),                                                   # no launches
    (dict(launch_src=[((0, 1, 1), (4, 1, 1), (8,))]), "ARG"),                       # zero grid dimension
    (dict(launch_src=[((1, 1, 1), (4, 1, 1), ())]), "ARG"),                          # scalar count mismatch
    (dict(launch_src=[((1, 1, 1), (4097, 1, 1), (8,))]), "LIMIT"),                  # > 4096 threads per block
    (dict(launch_src=[((2048, 1024, 1), (1, 1, 1), (8,))]), "LIMIT"),               # > 2^20 blocks
    (dict(launch_src=[((1, 1, 1), (4, 1, 1), (8,))], bits=33), "ARG"),
    (dict(launch_src=[((1, 1, 1), (4, 1, 1), (8,))], input_mode=7), "ARG"),
    (dict(launch_src=[((1, 1, 1), (4, 1, 1), (8,))], n_seeds=1, rank=2, world=2), "ARG"),
])
def test_argument_and_limit_errors(env, W, space, code):  # noqa: F811
    pgvc, torch = env
    k = pgvc.load_ir(W.subject("reduce1"))
    with pytest.raises(pgvc.PgError) as e:
        pgvc.check_races(k, pgvc.Space(**space))
    assert e.value.code == getattr(pgvc, "PG_E_" + code)


def test_shared_budget_limit(env):  # noqa: F811
    pgvc, torch = env
    k = pgvc.load_ir("kernel big(global out int o[1], unsigned n) { shared int s[n]; s[tid.x] = 1; sync; "
                     "o[0] = s[0]; }")
    with pytest.raises(pgvc.PgError) as e:
        pgvc.check_races(k, pgvc.Space([((1, 1, 1), (4, 1, 1), (1 << 20,))]))
    assert e.value.code == pgvc.PG_E_LIMIT


def test_record_buffer_truncation(env, oracle, W):  # noqa: F811
    # C1 non-square launches fail: cap the copy and the run's record buffer
    pgvc, torch = env
    ls = W.c1_launches()[:60]
    s, t = _irs(pgvc, W, "naive_transpose", "optimized_transpose")
    full, summ = pgvc.check_equiv(s, t, pgvc.Space(ls, n_seeds=4)).collect()
    assert summ["n_records"] == len(full) > 10
    part, summ2 = pgvc.check_equiv(s, t, pgvc.Space(ls, n_seeds=4)).collect(cap=10)
    assert part == full[:10] and summ2["n_records"] == summ["n_records"]
    capped, summ3 = pgvc.check_equiv(s, t, pgvc.Space(ls, n_seeds=4, max_cex=7)).collect()
    assert capped == full[:7] and summ3["first_key"] == summ["first_key"]


def test_one_thread_one_block(env, oracle, W):  # noqa: F811
    # the degenerate launch: 1 block of 1 thread (B = N = 1)
    ref, recs, summ, _ = run_pair(env, oracle, W.subject("reduce0"), W.subject("reduce2"),
                                  [W.reduce_launch("reduce0", 1, 1)], [W.reduce_launch("reduce2", 1, 1)], n_seeds=5)
    assert_same(ref, recs, summ)
    assert summ["instances"] == 5 * 2 * 1 * 2


def test_largest_block_races_mode(env, oracle, W):  # noqa: F811
    # 4096 emulated threads in one block (4 virtual threads per lane) with races and OOB
    text = ("kernel wide(global inout int a[4096]) { shared int s[4096]; s[tid.x] = a[tid.x]; sync; "
            "a[tid.x] = s[(tid.x * 3) % 4096] + s[tid.x + 1]; s[tid.x ^ 1] = tid.x; }")
    ref, recs, summ, _ = run_pair(env, oracle, text, None, [((1, 1, 1), (4096, 1, 1), ())], mode=1, n_seeds=2)
    assert_same(ref, recs, summ)
    assert summ["n_fail"] == 2


def test_repeated_and_interleaved_checks(env, oracle, W):  # noqa: F811
    # plans are cached per (kernels, space): interleave two spaces and re-run; results identical
    pgvc, torch = env
    s, t = _irs(pgvc, W, "reduce2", "reduce2_obo")
    a = pgvc.Space([W.reduce_launch("reduce2", 64, 16)], n_seeds=3)
    b = pgvc.Space([W.reduce_launch("reduce2", 8, 2), W.reduce_launch("reduce2", 16, 4)], n_seeds=2, seed_base=9)
    first = [pgvc.check_equiv(s, t, sp).collect() for sp in (a, b)]
    again = [pgvc.check_equiv(s, t, sp).collect() for sp in (b, a, b)]
    assert again[1] == first[0] and again[0] == first[1] and again[2] == first[1]


@pytest.mark.parametrize("T", [2, 48, 512])
def test_round_limit(env, oracle, T):  # noqa: F811
    # X19 round limit: 70000 barrier rounds; every live thread stops at round 0xFFFE with a
    # LIMIT record, as in the oracle (the optimistic pass flags, the exact re-run records)
    k = """
    kernel spin_sync(global out int o[n], unsigned n) {
      for (unsigned i = 0; i < 70000; i++) { sync; }
      o[bid.x * bdim.x + tid.x] = 1;
    }
    """
    ls = [((2, 1, 1), (T, 1, 1), (2 * T,))]
    ref, recs, summ, _ = run_pair(env, oracle, k, None, ls, mode=1, n_seeds=2)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][9] == 2 * 2 * T
