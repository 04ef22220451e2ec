"""GPU <-> oracle parity of property mode (pg_check_property):
a kernel against its post-condition kernel (subjects/post_*.pgk), bit-exact records,
counts and first-witness keys.  The oracle side runs oracle.check with the launches
include/pgvc.h says the library derives (workloads.property_launches)."""
import pytest

from test_gpu_parity import assert_same

pytestmark = pytest.mark.gpu

POST_SCALARS = {"post_reduce": 5, "post_scan": 5, "post_transpose": 6, "post_scalar_prod": 6}


@pytest.fixture(scope="module")
def env(oracle, W):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_lig12_b200 import build, pgvc
    build.build()
    return pgvc, torch


def run_prop(env, oracle, W, kernel, post, ls, n_seeds=3, **kw):
    pgvc, torch = env
    lt = W.property_launches(ls, POST_SCALARS[post])
    ref = oracle.check(W.subject(kernel), W.subject(post), ls, lt, n_seeds=n_seeds, cap=1 << 20, **kw)
    sp = pgvc.Space(ls, None, n_seeds=n_seeds, stream=torch.cuda.current_stream().cuda_stream, **kw)
    run = pgvc.check_property(pgvc.load_ir(W.subject(kernel)), pgvc.load_ir(W.subject(post)), sp)
    recs, summ = run.collect(cap=1 << 20)
    assert_same(ref, recs, summ)
    return summ


@pytest.mark.parametrize("kernel", ["reduce0", "reduce1", "reduce2", "reduce2_obo", "reduce3", "reduce4",
                                    "reduce5", "reduce6", "reduce0_lit"])
def test_property_reductions(env, oracle, W, kernel):
    pts = [(N, B) for B in (1, 2, 4, 16, 64) for N in (B, 4 * B, 256) if N >= B and N % B == 0]
    ls = [W.reduce_launch(kernel, N, B) for N, B in pts if not (kernel in W.REDUCE_HALF and B < 2)]
    summ = run_prop(env, oracle, W, kernel, "post_reduce", ls)
    if kernel in ("reduce0", "reduce1", "reduce2", "reduce3", "reduce6"):
        assert summ["n_fail"] == 0


def test_property_scans(env, oracle, W):
    for k in ("prescan", "prescan_nobarrier"):
        ls = [W.scan_launch(k, n, B) for (n, B) in [(2, 1), (8, 2), (32, 4), (64, 8), (128, 64)]]
        summ = run_prop(env, oracle, W, k, "post_scan", ls)
        assert (summ["n_fail"] == 0) == (k == "prescan")


def test_property_transposes(env, oracle, W):
    ls = W.c1_launches()[::7]
    for k in ("naive_transpose", "optimized_transpose"):
        summ = run_prop(env, oracle, W, k, "post_transpose", ls, n_seeds=2)
        assert (summ["n_fail"] == 0) == (k == "naive_transpose")


def test_property_rejects_tgt_and_scalar_shortfall(env, W):
    pgvc, torch = env
    k = pgvc.load_ir(W.subject("reduce1"))
    post = pgvc.load_ir(W.subject("post_transpose"))   # wants 6 scalars; a reduction launch gives 5
    with pytest.raises(pgvc.PgError):
        pgvc.check_property(k, post, pgvc.Space([W.reduce_launch("reduce1", 8, 4)]))
    with pytest.raises(ValueError):
        pgvc.check_property(k, post, pgvc.Space([W.reduce_launch("reduce1", 8, 4)], [W.reduce_launch("reduce1", 8, 4)]))
