"""Oracle pins for the transpose pair (PAPER.md L122-L171, L601-L657, L769-L774,
Table II)."""
import numpy as np
import pytest

KIND = {"OOB": 1, "RACE_WW": 2, "MISMATCH": 5}


@pytest.fixture(scope="module")
def c1_run(oracle, W):
    w = W.c1()
    r = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=8, cap=1 << 18)
    return w, r


FAILING = {0, 1, 2, 3, 4, 5, 9}


def test_square_blocks_equivalent_nonsquare_not(oracle, W, c1_run):
    # P2(i)/(ii), L639-L651: equivalent iff bdim.x == bdim.y; every non-square launch fails
    w, r = c1_run
    failing = {}
    for rec in r["records"]:
        d = dict(zip(oracle.REC_FIELDS, rec))
        if d["kind"] in FAILING:
            failing.setdefault(d["launch"], set()).add(d["seed_idx"])
    sq = [i for i, l in enumerate(w.launch_src) if l.bdim[0] == l.bdim[1]]
    nsq = [i for i, l in enumerate(w.launch_src) if l.bdim[0] != l.bdim[1]]
    assert len(w.launch_src) == 1089 and len(sq) == 361 and len(nsq) == 728
    assert not any(i in failing for i in sq)
    assert all(failing.get(i) == set(range(8)) for i in nsq)
    assert r["counts"][12] == 728 * 8


def test_oob_exactly_when_by_gt_bx(oracle, W, c1_run):
    # block[bdim.x][bdim.x+1] holds block[tid.y][tid.x] only if bdim.y <= bdim.x (L155, L161)
    w, r = c1_run
    oob = {dict(zip(oracle.REC_FIELDS, x))["launch"] for x in r["records"] if x[2] == KIND["OOB"]}
    want = {i for i, l in enumerate(w.launch_src) if l.bdim[1] > l.bdim[0]}
    assert oob == want and len(want) == 364


def test_first_witness(oracle, W, c1_run):
    # smallest witnessing n: n = 2, bdim = (2,1), gdim = (1,1), width = 2, height = 1; odata[1]
    # is written with idata[1] by the naive kernel and left initial by the optimized one
    w, r = c1_run
    first = r["first_key"][0]
    li = first >> 45
    l = w.launch_src[li]
    assert (l.threads, l.bdim, l.gdim, l.scalars) == (2, (2, 1, 1), (1, 1, 1), (2, 1))
    (rec,) = [x for x in r["records"] if x[0] == first]
    d = dict(zip(oracle.REC_FIELDS, rec))
    assert d["kind"] == KIND["MISMATCH"] and d["addr"] == 1 and d["tid_a"] == 1 and d["tid_b"] == 0xFFFFFFFF
    init, _, _ = oracle.exec_kernel(W.subject("naive_transpose"), l, 0)
    assert d["val_a"] == int(init[0][1])          # gid 0 = idata (sorted names)


def test_closed_form_postcondition(oracle, W):
    # P2(iv), L133-L134: odata[i*height + j] == idata[j*width + i] for i < width, j < height
    for l in W.c1_launches():
        if l.bdim[0] != l.bdim[1] or l.threads not in (1, 4, 16, 36, 64, 144, 256):
            continue
        wd, ht = l.scalars
        for name in ("naive_transpose", "optimized_transpose"):
            _, fin, counts = oracle.exec_kernel(W.subject(name), l, 3)
            idata, odata = fin[0].reshape(ht, wd), fin[1].reshape(wd, ht)
            assert (odata == idata.T).all()
            assert sum(counts[1:9]) == counts[1 + 8] == 0   # no failing kind, no UNINIT


def test_writer_relation_t1_is_transposed_t2(oracle, W):
    # P2(iii), L619-L627: in round 2 of OptimizedTranspose the read block[t2.x][t2.y] is supplied by
    # the round-1 write of thread t1 = (t2.y, t2.x) of the same block (constraint t2.x = t1.y /\ t2.y = t1.x)
    for b in (2, 3, 4):
        l = ((2, 2, 1), (b, b, 1), (2 * b, 2 * b))
        rows = oracle.dataflow(W.subject("optimized_transpose"), l, 5)
        shared_reads = [dict(zip(oracle.DF_FIELDS, r)) for r in rows if r[4] == 0x100]
        assert len(shared_reads) == 4 * b * b
        T = b * b
        for d in shared_reads:
            t2 = d["gtid"] - d["block"] * T
            t2x, t2y = t2 % b, t2 // b
            assert d["round"] == 1 and d["src_kind"] == 1
            assert (d["w_block"], d["w_round"]) == (d["block"], 0)
            assert d["w_gtid"] - d["block"] * T == t2x * b + t2y   # t1 = (x = t2.y, y = t2.x)


def test_unique_writer_under_square_blocks(oracle, W):
    # P2(v), L769-L774: under valid configurations every output cell has exactly one writer,
    # so the quantified "no writer" formula is never needed
    ls = [l for l in W.c1_launches() if l.bdim[0] == l.bdim[1]][::7]
    for name in ("naive_transpose", "optimized_transpose"):
        r = oracle.check(W.subject(name), None, ls, mode=1, checks=oracle.RACE | oracle.OOB, n_seeds=2)
        assert r["counts"][1:11] == [0] * 10
        for l in ls:
            rows = oracle.dataflow(W.subject("naive_transpose"), l, 1)
            assert all(r[6] == 0 for r in rows)   # naive reads only idata, never written


def test_table2_star_pattern(oracle, W):
    # Table II: starred (not equivalent) exactly when n is not a perfect square
    golden = []
    with open(__import__("os").path.join(__import__("os").path.dirname(__file__), "golden",
                                         "table2_transpose_verdicts.txt")) as f:
        for line in f:
            if line.strip() and not line.startswith("#"):
                n, star = line.split()
                golden.append((int(n), int(star)))
    src, tgt = W.subject("naive_transpose"), W.subject("optimized_transpose")
    for n, star in golden:
        shapes = [(bx, n // bx) for bx in range(1, n + 1) if n % bx == 0]
        ls = []
        for bx, by in shapes:
            ls.append(((1, 1, 1), (bx, by, 1), (bx, by)))
            ls.append(((2, 2, 1), (bx, by, 1), (2 * bx, 2 * by)))
        r = oracle.check(src, tgt, ls, ls, n_seeds=2)
        fail_launch = {x[3] for x in r["records"] if x[2] in FAILING}
        equivalent_shapes = [shapes[i // 2] for i in range(len(ls)) if i not in fail_launch]
        assert bool(star) == (len(equivalent_shapes) == 0)
        assert all(bx == by for bx, by in equivalent_shapes)
