"""Property mode on the oracle: the post-condition kernels
subjects/post_*.pgk against the closed forms the paper states, and the verdicts of
kernel-vs-post-condition checks.

Pins:
* post_reduce computes sum_{i<B} in[b*B + i] mod 2^32 (reading X11),
  checked against numpy on the oracle's own initial arrays;
* post_scan computes the block-local exclusive prefix sum (L471-L472, X11);
* post_transpose computes odata[i*h + j] = idata[j*w + i] (L133-L134);
* correct kernels satisfy their post-condition; the literal L825 loop (X10) first
  fails at bdim = 4, reduce2_obo and the barrier-less scan fail."""
import numpy as np

POST_SCALARS = {"post_reduce": 5, "post_scan": 5, "post_transpose": 6}


def post_run(oracle, W, post, launch, seed):
    pl = W.property_launches([launch], POST_SCALARS[post])[0]
    init, fin, counts = oracle.exec_kernel(W.subject(post), pl, seed)
    return init, fin, counts


def test_post_reduce_closed_form(oracle, W):
    for N, B in [(8, 4), (64, 16), (48, 16), (32, 1)]:
        for seed in (0, 3):
            init, fin, counts = post_run(oracle, W, "post_reduce", W.reduce_launch("reduce1", N, B), seed)
            x = init[0].astype(np.uint64)           # g_idata (gid 0), g_odata (gid 1)
            want = (x.reshape(N // B, B).sum(axis=1) % (1 << 32)).astype(np.uint32)
            assert (fin[1] == want).all()
            assert counts[2] == 0                    # no failing record in a one-thread run


def test_post_scan_closed_form(oracle, W):
    for n, B in [(8, 2), (32, 4), (64, 32)]:
        init, fin, _ = post_run(oracle, W, "post_scan", W.scan_launch("prescan", n, B), 2)
        x = init[0].astype(np.uint64)                # g_idata sorts before g_odata
        m = 2 * B
        want = np.zeros(n, dtype=np.uint64)
        for b in range(n // m):
            want[b * m + 1:(b + 1) * m] = np.cumsum(x[b * m:(b + 1) * m - 1])
        assert (fin[1] == (want % (1 << 32)).astype(np.uint32)).all()


def test_post_transpose_closed_form(oracle, W):
    for (gx, gy, bx, by) in [(2, 1, 2, 3), (1, 1, 4, 4), (3, 2, 2, 2)]:
        w, h = gx * bx, gy * by
        l = W.Launch((gx, gy, 1), (bx, by, 1), (w, h))
        init, fin, _ = post_run(oracle, W, "post_transpose", l, 1)
        idata = init[0].reshape(h, w)                # idata < odata
        assert (fin[1].reshape(w, h) == idata.T).all()


def check_prop(oracle, W, kernel, post, launches, n_seeds=2):
    lt = W.property_launches(launches, POST_SCALARS[post])
    return oracle.check(W.subject(kernel), W.subject(post), launches, lt, n_seeds=n_seeds)


def fails(res):
    return res["counts"][12]


def test_reductions_satisfy_post(oracle, W):
    for k in ("reduce0", "reduce1", "reduce2", "reduce3", "reduce6"):
        ls = [W.reduce_launch(k, N, B) for (N, B) in [(16, 4), (64, 16), (256, 64), (32, 32)]
              if (k not in W.REDUCE_HALF or B >= 2)]
        assert fails(check_prop(oracle, W, k, "post_reduce", ls)) == 0, k


def test_literal_loop_fails_first_at_bdim_4(oracle, W):
    # X10 / P3(v): the loop header as printed at L825 sums a0 + a2 at bdim = 4
    ls = [W.reduce_launch("reduce0_lit", B, B) for B in (1, 2, 4, 8)]
    res = check_prop(oracle, W, "reduce0_lit", "post_reduce", ls)
    assert fails(res) > 0
    assert res["first_key"][0] >> 45 == 2          # launch index 2: bdim = 4 (X16 key)


def test_obo_mutant_fails_post(oracle, W):
    ls = [W.reduce_launch("reduce2_obo", N, B) for (N, B) in [(2, 2), (8, 4)]]
    assert fails(check_prop(oracle, W, "reduce2_obo", "post_reduce", ls)) > 0


def test_scans_against_post(oracle, W):
    ls = [W.scan_launch("prescan", n, B) for (n, B) in [(8, 2), (32, 4), (64, 8)]]
    assert fails(check_prop(oracle, W, "prescan", "post_scan", ls)) == 0
    ls = [W.scan_launch("prescan_nobarrier", n, B) for (n, B) in [(8, 2), (32, 4)]]
    assert fails(check_prop(oracle, W, "prescan_nobarrier", "post_scan", ls)) > 0


def test_transposes_against_post(oracle, W):
    ls = W.c1_launches()[:120]
    assert fails(check_prop(oracle, W, "naive_transpose", "post_transpose", ls, 1)) == 0
    res = check_prop(oracle, W, "optimized_transpose", "post_transpose", ls, 1)
    square = sum(1 for l in ls if l.bdim[0] == l.bdim[1])
    assert res["counts"][12] == len(ls) - square    # every non-square launch fails (P2 ii)
