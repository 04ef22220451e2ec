"""GPU parity of multi-kernel sequences (pg_check_equiv_seq, GKLEE's
multi-kernel programs PAPER.md L62-L63): the phases of a side share their global buffers,
records per phase, final buffers compared - bit-exact against oracle.check_seq."""
import pytest

from test_gpu_parity import assert_same, env, ir  # noqa: F401  (env: fixture)

pytestmark = pytest.mark.gpu


def _gpu(env, W, src, tgt, sl, tl, n_seeds, seed_base=0, texts=None):
    pgvc, torch = env
    t = texts or {}
    sp = pgvc.Space(sl[0], n_seeds=n_seeds, seed_base=seed_base, stream=torch.cuda.current_stream().cuda_stream)
    run = pgvc.check_equiv_seq([ir(pgvc, t.get(n) or W.subject(n)) for n in src],
                               [ir(pgvc, t.get(n) or W.subject(n)) for n in tgt], sl, tl, sp)
    return run.collect(cap=1 << 20)


@pytest.mark.parametrize("first", ["reduce0", "reduce2_obo", "reduce1"])
def test_two_pass_reduction(env, oracle, W, first):
    w = W.reduce_two_pass(max_log_n=12, max_log_b=8, first=first)
    ref = oracle.check_seq([W.subject(n) for n in w.src], [W.subject(n) for n in w.tgt], w.src_launches,
                           w.tgt_launches, n_seeds=3, seed_base=5, cap=1 << 20)
    recs, summ = _gpu(env, W, w.src, w.tgt, w.src_launches, w.tgt_launches, 3, seed_base=5)
    assert_same(ref, recs, summ)


def test_second_phase_alone_and_reversed_sides(env, oracle, W):
    w = W.reduce_two_pass(max_log_n=9, max_log_b=4)
    ref = oracle.check_seq([W.subject("reduce0_pass2")], [W.subject("sum_serial")], [w.src_launches[1]],
                           w.tgt_launches, n_seeds=2, cap=1 << 20)
    recs, summ = _gpu(env, W, ["reduce0_pass2"], ["sum_serial"], [w.src_launches[1]], w.tgt_launches, 2)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][5] > 0
    # the sequence as the target side: records of its phases are kernels 1 and 2
    ref = oracle.check_seq([W.subject("sum_serial")], [W.subject(n) for n in w.src], w.tgt_launches,
                           w.src_launches, n_seeds=2, cap=1 << 20)
    recs, summ = _gpu(env, W, ["sum_serial"], w.src, w.tgt_launches, w.src_launches, 2)
    assert_same(ref, recs, summ)


def test_three_phase_sequence_with_races(env, oracle, W):
    # block sums with the racy barrier-free scan as a middle phase: races of phase 1 recorded as
    # kernel 1, the two sides' shared buffer g_sum compared
    w = W.reduce_two_pass(max_log_n=8, max_log_b=3)
    mid = """
    kernel touch(global inout int g_odata[m], unsigned m) {
      shared int s[bdim.x];
      s[tid.x] = g_odata[tid.x];
      if (tid.x > 0) { g_odata[tid.x] = s[tid.x] + s[tid.x - 1]; }
    }
    """
    texts = {"touch": mid}
    ml = [W.Launch((1, 1, 1), (l.bdim[0], 1, 1), (l.scalars[0],)) for l in w.src_launches[1]]
    src = ["reduce0", "touch", "reduce0_pass2"]
    sl = [w.src_launches[0], ml, w.src_launches[1]]
    ref = oracle.check_seq([W.subject("reduce0"), mid, W.subject("reduce0_pass2")], [W.subject("sum_serial")],
                           sl, w.tgt_launches, n_seeds=2, cap=1 << 20)
    recs, summ = _gpu(env, W, src, ["sum_serial"], sl, w.tgt_launches, 2, texts=texts)
    assert_same(ref, recs, summ)
