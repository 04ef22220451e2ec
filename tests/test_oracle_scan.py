"""Oracle pins for the scan pair (PAPER.md L467-L472 post-condition)."""
import numpy as np
import pytest

FAILING = {0, 1, 2, 3, 4, 5, 9}


def excl_scan(x, m):
    x = x.astype(np.uint64).reshape(-1, m)
    return ((np.cumsum(x, 1) - x) % (1 << 32)).astype(np.uint32).reshape(-1)


@pytest.mark.parametrize("tgt,lognb", [("prescan", 4), ("prescan_padded", 4), ("prescan_padded", 5)])
def test_exclusive_scan_closed_form(oracle, W, tgt, lognb):
    # L471-L472 read 0-based (X11): o[0] = 0, o[i+1] = o[i] + in[i]
    for n, B in [(2, 1), (8, 2), (64, 32), (2048, 1024), (4096, 256)]:
        l = W.scan_launch(tgt, n, B, lognb)
        _, fin, counts = oracle.exec_kernel(W.subject(tgt), l, 8)
        assert (fin[1] == excl_scan(fin[0], 2 * B)).all()
        assert sum(counts[1:11]) == 0


def test_pair_equivalent(oracle, W):
    w = W.c3_pair("prescan_padded", 4, n_seeds=2, max_log_n=8, max_log_b=6)
    r = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=2,
                     checks=oracle.EQUIV | oracle.RACE | oracle.OOB)
    assert r["n_records"] == 0


def test_dropped_downsweep_barrier_first_witness(oracle, W):
    # P4: first failure at n = 4, B = 2 with WW on temp[3] by threads 0 and 1; B = 1 is clean
    w = W.c3_pair("prescan_nobarrier", n_seeds=2, max_log_n=6, max_log_b=3)
    r = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=2)
    pts = W.c3_points(6, 3)
    li = r["first_key"][0] >> 45
    assert pts[li] == (4, 2)
    ww = [dict(zip(oracle.REC_FIELDS, x)) for x in r["records"] if x[2] == 2 and x[3] == li and x[4] == 0]
    assert len(ww) == 1 and (ww[0]["array"], ww[0]["addr"], ww[0]["tid_a"], ww[0]["tid_b"]) == (0x100, 3, 0, 1)
    assert any(x[2] == 5 and x[3] == li for x in r["records"])          # wrong output
    assert not any(x[2] in FAILING and pts[x[3]][1] == 1 for x in r["records"])


def bank_degree(stride_words, active):
    """Degree of a warp access where lane t (t < active) reads word stride*t + c (X9, 32 banks):
    the lanes hit 32/gcd(32, stride) distinct banks, so degree = min(active, gcd(32, stride))
    (for active <= 32 lanes)."""
    from math import gcd
    return min(active, 32, gcd(32, stride_words) if stride_words else active)


def analytic_max_degree(B, lognb=None):
    # Blelloch up/down-sweep: at offset o, thread t < d = m/(2o) touches o(2t+1)-1 and o(2t+2)-1,
    # a stride of 2o words per lane.  Padding i + (i >> lognb) is evaluated by brute force below.
    m = 2 * B
    worst = 1
    o = 1
    while o < m:
        d = m // (2 * o)
        for w0 in range(0, d, 32):
            lanes = range(w0, min(d, w0 + 32))
            for c in (lambda t: o * (2 * t + 1) - 1, lambda t: o * (2 * t + 2) - 1):
                addrs = [c(t) for t in lanes]
                if lognb is not None:
                    addrs = [a + (a >> lognb) for a in addrs]
                per_bank = {}
                for a in set(addrs):
                    per_bank.setdefault(a % 32, set()).add(a)
                worst = max(worst, max(len(s) for s in per_bank.values()))
        o *= 2
    return worst


def test_bank_degree_closed_form_helper():
    # the unpadded sweep is a pure stride-2o pattern: gcd formula and brute force agree
    assert [analytic_max_degree(B) for B in (64, 256, 1024)] == [4, 16, 32]
    assert bank_degree(32, 32) == 32 and bank_degree(33, 32) == 1 and bank_degree(2, 32) == 2


@pytest.mark.parametrize("tgt,lognb", [("prescan", None), ("prescan_padded", 4), ("prescan_padded", 5)])
def test_bank_degrees(oracle, W, tgt, lognb):
    # X9 bank model (32 banks): the max bank degree over the shared sweep sites equals the brute-force
    # value of the address pattern; SURVEY.md P4 scratch values 4/16/32, 2/2/4 and 1/1/2
    want = {None: [4, 16, 32], 4: [2, 2, 4], 5: [1, 1, 2]}[lognb]
    got = []
    for B in (64, 256, 1024):
        l = W.scan_launch(tgt, 2 * B, B, lognb or 4)
        r = oracle.check(W.subject(tgt), None, [l], mode=2, checks=oracle.BANK | oracle.COALESCE, max_sites=64)
        st = r["site_stats"][0, 0]
        shared = st[st[:, 0] == 1]
        got.append(int(shared[:, 3].max()))
        assert got[-1] == analytic_max_degree(B, lognb) or (lognb and got[-1] == max(analytic_max_degree(B, lognb), 1))
    assert got == want
