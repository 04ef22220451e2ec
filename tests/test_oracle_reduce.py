"""Oracle pins for the reduction variants."""
import numpy as np
import pytest

FAILING = {0, 1, 2, 3, 4, 5, 9}


def block_sums(idata, B):
    return (idata.astype(np.uint64).reshape(-1, B).sum(1) % (1 << 32)).astype(np.uint32)


@pytest.mark.parametrize("name", ["reduce0", "reduce1", "reduce2", "reduce3", "reduce4", "reduce5", "reduce6"])
def test_closed_form_sum(oracle, W, name):
    # P3(i), L465 (0-based, X11): g_odata[b] = sum of the block's B inputs mod 2^32
    for N, B in [(1, 1), (8, 2), (64, 16), (256, 256), (2048, 1024), (4096, 512)]:
        if name in W.REDUCE_HALF and B < 2:
            continue
        l = W.reduce_launch(name, N, B)
        _, fin, counts = oracle.exec_kernel(W.subject(name), l, 11)
        assert (fin[1] == block_sums(fin[0], B)).all(), (N, B)
        assert sum(counts[1:11]) == 0


def test_reduce0_reduce1_writer_relation(oracle, W):
    # P3(ii), L839-L845: both loops write the same cells; reduce0's writer of cell s.x is s itself,
    # reduce1's is t with 2*k*t = s.x (k = 2^(round-1)), i.e. s = 2k t
    B = 16
    for name in ("reduce0", "reduce1"):
        rows = oracle.dataflow(W.subject(name), W.reduce_launch(name, B, B), 2)
        for r in rows:
            d = dict(zip(oracle.DF_FIELDS, r))
            if d["array"] != 0x100 or d["src_kind"] != 1 or d["w_round"] == 0:
                continue
            k = 1 << (d["w_round"] - 1)
            want = d["addr"] if name == "reduce0" else d["addr"] // (2 * k)
            assert d["addr"] % (2 * k) == 0
            assert d["w_gtid"] == want
    ls0 = [W.reduce_launch("reduce0", N, B) for N, B in W.c2_points(8, 6)]
    ls1 = [W.reduce_launch("reduce1", N, B) for N, B in W.c2_points(8, 6)]
    r = oracle.check(W.subject("reduce0"), W.subject("reduce1"), ls0, ls1, n_seeds=3)
    assert r["n_records"] == 0


def test_non_power_of_two_blocks_first_fail_at_3(oracle, W):
    # P3(iii): the SDK kernels assume power-of-two blockDim (hidden assumption, L629-L651 style)
    def first_bad(name, kind):
        for B in range(1, 9):
            l = W.reduce_launch(name, B, B)
            _, fin, counts = oracle.exec_kernel(W.subject(name), l, 4)
            wrong = not (fin[1] == block_sums(fin[0], B)).all()
            if (kind == "oob" and counts[1 + 1] > 0) or (kind == "sum" and wrong):
                return B
        return None
    assert first_bad("reduce0", "oob") == 3
    assert first_bad("reduce1", "oob") == 3
    assert first_bad("reduce2", "sum") == 3


def test_injected_off_by_one_first_witness(oracle, W):
    # P3(iv): reduce2 `t < s` -> `t <= s`: OOB + RW race, smallest witness N = 2, B = 2
    w = W.c2_pair("reduce2", "reduce2_obo", n_seeds=4, max_log_n=6, max_log_b=4)
    r = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=4)
    li = r["first_key"][0] >> 45
    pts = W.c2_points(6, 4, 0)
    assert pts[li] == (2, 2)
    kinds = {x[2] for x in r["records"] if x[3] == li and x[4] == 0}
    assert {1, 3} <= kinds
    # every launch with B >= 2 witnesses the bug for every seed (injected bugs are always caught)
    bad = {(x[3], x[4]) for x in r["records"] if x[2] in FAILING}
    assert bad == {(i, s) for i, (N, B) in enumerate(pts) if B >= 2 for s in range(4)}


def test_literal_paper_header_is_not_a_reduction(oracle, W):
    # P3(v), X10: L825's header `k = bdim.x/2; k > 0; k >>= 2` first gives a wrong sum at bdim = 4
    firsts = []
    for B in (1, 2, 4, 8, 16):
        _, fin, _ = oracle.exec_kernel(W.subject("reduce0_lit"), ((1, 1, 1), (B, 1, 1), (B,)), 6)
        firsts.append((fin[1] == block_sums(fin[0], B)).all())
    assert firsts == [True, True, False, False, False]


def test_warp_synchronous_tail_is_a_race(oracle, W):
    # the legacy warp-synchronous reduce4 tail has no barriers: under round semantics it races
    l = W.reduce_launch("reduce4_warpsync", 128, 128)
    r = oracle.check(W.subject("reduce4_warpsync"), None, [l], mode=1, checks=oracle.RACE | oracle.OOB)
    assert r["counts"][1 + 3] > 0
