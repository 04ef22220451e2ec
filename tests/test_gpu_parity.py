"""GPU <-> oracle parity (bit-exact): identical record lists (canonical order, every
field), identical per-kind counts, instance counts and first-witness keys.
Calls go through the C ABI (pgvc binding).  Needs a B200: `pytest -m gpu`."""
import pytest

pytestmark = pytest.mark.gpu

KW_ORACLE = ("n_seeds", "seed_base", "input_mode", "input_range", "bits", "checks", "bank_model", "rank", "world")


@pytest.fixture(scope="module")
def env(oracle, W):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_lig12_b200 import build, pgvc
    build.build()
    return pgvc, torch


_ir_cache = {}


def ir(pgvc, text):
    if text not in _ir_cache:
        _ir_cache[text] = pgvc.load_ir(text)
    return _ir_cache[text]


def run_pair(env, oracle, src, tgt, ls, lt=None, mode=0, max_sites=0, **kw):
    pgvc, torch = env
    lt = lt if lt is not None else (ls if tgt else None)
    okw = {k: v for k, v in kw.items() if k in KW_ORACLE}
    if mode == 1:       # pg_check_races: checks = RACE | OOB
        okw["checks"] = oracle.RACE | oracle.OOB
    elif mode == 2:     # pg_check_banks: checks = BANK | COALESCE
        okw["checks"] = oracle.BANK | oracle.COALESCE
    ref = oracle.check(src, tgt, ls, lt, mode=mode, max_sites=max_sites, cap=1 << 20, **okw)
    sp = pgvc.Space(ls, lt, stream=torch.cuda.current_stream().cuda_stream, **kw)
    if mode == 0:
        run = pgvc.check_equiv(ir(pgvc, src), ir(pgvc, tgt), sp)
    elif mode == 1:
        run = pgvc.check_races(ir(pgvc, src), sp)
    else:
        run = pgvc.check_banks(ir(pgvc, src), sp)
    recs, summ = run.collect(cap=1 << 20)
    stats = run.site_stats(max_sites) if max_sites else None
    return ref, recs, summ, stats


def assert_same(ref, recs, summ):
    assert summ["instances"] == ref["counts"][0]
    assert summ["per_kind"] == ref["counts"][1:11]
    assert summ["n_records"] == ref["n_records"]
    assert summ["n_fail"] == ref["counts"][12]
    assert summ["first_key"] == ref["first_key"][0]
    assert summ["first_key_kind"] == ref["first_key"][1:11]
    if recs != ref["records"]:
        for a, b in zip(recs, ref["records"]):
            if a != b:
                raise AssertionError("first differing record:\n gpu    %s\n oracle %s" % (a, b))
        raise AssertionError("record list lengths differ: %d vs %d" % (len(recs), len(ref["records"])))


# ---------------------------------------------------------------- C1 (configs[0]) in full
def test_c1_full(env, oracle, W):
    w = W.c1(n_seeds=64)
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, n_seeds=64)
    assert_same(ref, recs, summ)
    assert summ["instances"] == 85849 * 3 * 64
    assert summ["n_fail"] == 728 * 64


def test_c1_ragged_sizes(env, oracle, W):
    ls = W.c1_launches(ragged=True)[::5]
    ref, recs, summ, _ = run_pair(env, oracle, W.subject("naive_transpose"), W.subject("optimized_transpose"), ls,
                                  n_seeds=4, seed_base=1000)
    assert_same(ref, recs, summ)


def test_c1_sharded_union(env, oracle, W):
    ls = W.c1_launches()[:200]
    src, tgt = W.subject("naive_transpose"), W.subject("optimized_transpose")
    full = run_pair(env, oracle, src, tgt, ls, n_seeds=6)
    parts = [run_pair(env, oracle, src, tgt, ls, n_seeds=6, rank=r, world=3) for r in range(3)]
    for ref, recs, summ, _ in parts:
        assert_same(ref, recs, summ)
    merged = sorted(r for p in parts for r in p[1])
    assert merged == full[1]
    assert sum(p[2]["instances"] for p in parts) == full[2]["instances"]


# ---------------------------------------------------------------- C2 reductions
@pytest.mark.parametrize("pair", [("reduce0", "reduce1"), ("reduce0", "reduce2"), ("reduce0", "reduce3"),
                                  ("reduce0", "reduce4"), ("reduce0", "reduce5"), ("reduce0", "reduce6"),
                                  ("reduce2", "reduce2_obo")])
def test_c2_pairs_reduced_space(env, oracle, W, pair):
    w = W.c2_pair(*pair, n_seeds=3, max_log_n=10, max_log_b=10)
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt,
                                  n_seeds=3)
    assert_same(ref, recs, summ)


def test_c2_pairs_concurrent_streams(env, oracle, W):
    """bench.py's launch configuration: the seven C2 pairs enqueued together, one stream
    each (forked from and joined into one stream), each pair writing its own key/count
    rows; every pair must still equal the oracle."""
    pgvc, torch = env
    ws = W.c2(n_seeds=3, max_log_n=9, max_log_b=9)
    main = torch.cuda.current_stream()
    side = [torch.cuda.Stream() for _ in ws]
    keys = torch.empty(len(ws), 11, dtype=torch.int64, device="cuda")
    cnts = torch.empty(len(ws), 16, dtype=torch.int64, device="cuda")
    fork = torch.cuda.Event()
    fork.record(main)
    runs = []
    for i, w in enumerate(ws):
        side[i].wait_event(fork)
        sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=3, checks=w.checks, stream=side[i].cuda_stream,
                        first_key=keys[i], counts=cnts[i])
        runs.append(pgvc.check_equiv(ir(pgvc, W.subject(w.src)), ir(pgvc, W.subject(w.tgt)), sp))
    for st in side:
        main.wait_stream(st)
    torch.cuda.synchronize()
    for i, (w, run) in enumerate(zip(ws, runs)):
        recs, summ = run.collect(cap=1 << 20)
        ref = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=3,
                           checks=w.checks, cap=1 << 20)
        assert_same(ref, recs, summ)
        assert cnts[i][0].item() == ref["counts"][0]


def test_c2_full_size_launches(env, oracle, W):
    # BASELINE sizes: N = 2^16 with B = 1, 32, 1024, one seed each (oracle computes these one by one)
    for src, tgt in (("reduce0", "reduce6"), ("reduce2", "reduce2_obo")):
        pts = [(1 << 16, 1 << lb) for lb in (1, 5, 10)]
        ls = [W.reduce_launch(src, N, B) for N, B in pts]
        lt = [W.reduce_launch(tgt, N, B) for N, B in pts]
        ref, recs, summ, _ = run_pair(env, oracle, W.subject(src), W.subject(tgt), ls, lt, n_seeds=1, seed_base=77)
        assert_same(ref, recs, summ)


def test_c2_literal_header_and_warpsync(env, oracle, W):
    pts = W.c2_points(9, 8, 1)
    ls = [W.reduce_launch("reduce0", N, B) for N, B in pts]
    ref, recs, summ, _ = run_pair(env, oracle, W.subject("reduce0"), W.subject("reduce0_lit"), ls, n_seeds=2)
    assert_same(ref, recs, summ)
    lt = [W.reduce_launch("reduce4_warpsync", N, B) for N, B in pts]
    ref, recs, summ, _ = run_pair(env, oracle, W.subject("reduce4_warpsync"), None, lt, mode=1, n_seeds=2)
    assert_same(ref, recs, summ)


# ---------------------------------------------------------------- C3 scan
@pytest.mark.parametrize("tgt,lognb", [("prescan_padded", 4), ("prescan_padded", 5), ("prescan_nobarrier", 4)])
def test_c3_pairs(env, oracle, W, tgt, lognb):
    w = W.c3_pair(tgt, lognb, n_seeds=2, max_log_n=11, max_log_b=10)
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt,
                                  n_seeds=2, checks=31)
    assert_same(ref, recs, summ)


@pytest.mark.parametrize("name", ["prescan", "prescan_padded"])
def test_c3_bank_stats(env, oracle, W, name):
    ls = [W.scan_launch(name, n, B) for n, B in W.c3_points(11, 10)][::3]
    ref, recs, summ, stats = run_pair(env, oracle, W.subject(name), None, ls, mode=2, max_sites=48, n_seeds=2)
    assert_same(ref, recs, summ)
    assert (stats == ref["site_stats"]).all()


# ---------------------------------------------------------------- C4 bitonic
def test_c4_random_and_ties(env, oracle, W):
    for w in W.c4("rand", n_seeds=4, max_log_n=9) + W.c4("range", n_seeds=4, max_log_n=9):
        ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt,
                                      n_seeds=4, input_mode=w.input_mode, input_range=w.input_range)
        assert_same(ref, recs, summ)
        assert summ["n_fail"] == 0


def test_c4_exhaustive_01(env, oracle, W):
    for w in W.c4("bits", max_log_n=3):
        ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt,
                                      n_seeds=w.n_seeds, input_mode=1)
        assert_same(ref, recs, summ)


def test_c4_virtual_threads_4096(env, oracle, W):
    # bitonic_global at n = 4096 has 4096 threads in one block (> 1024): virtual threads
    for n in (2048, 4096):
        ls, lt = [W.bitonic_launch("bitonic_global", n)], [W.bitonic_launch("bitonic_shared", n)]
        ref, recs, summ, _ = run_pair(env, oracle, W.subject("bitonic_global"), W.subject("bitonic_shared"), ls, lt,
                                      n_seeds=1)
        assert_same(ref, recs, summ)


# ---------------------------------------------------------------- C5 (small sizes)
def test_c5_small(env, oracle, W):
    w = W.c5_transpose(n_seeds=2, sizes=(32, 64))
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, n_seeds=2)
    assert_same(ref, recs, summ)
    w = W.c5_matmul(n_seeds=2, sizes=(32, 64), K=64)
    ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, n_seeds=2)
    assert_same(ref, recs, summ)
    ls = [((2, 2, 1), (4, 4, 1), (K, 8, 8)) for K in (4, 8, 12)]
    ref, recs, summ, _ = run_pair(env, oracle, W.subject("matmul_tiled"), W.subject("matmul_tiled_nobarrier"), ls,
                                  n_seeds=2)
    assert_same(ref, recs, summ)


def test_c5_banks_and_coalescing(env, oracle, W):
    l = [((1, 1, 1), (32, 32, 1), (32, 32)), ((2, 2, 1), (32, 32, 1), (64, 64))]
    for name in ("naive_transpose", "optimized_transpose", "optimized_transpose_unpadded"):
        ref, recs, summ, stats = run_pair(env, oracle, W.subject(name), None, l, mode=2, max_sites=8, n_seeds=1)
        assert_same(ref, recs, summ)
        assert (stats == ref["site_stats"]).all()


# ---------------------------------------------------------------- semantics fixtures
FIXTURES = [
    ("kernel tw(global inout int v[2 * n], unsigned n) { unsigned i = 0; unsigned j = tid.x + n; v[i] = v[j] + tid.x; sync; v[tid.x]++; }",
     [((1, 1, 1), (4, 1, 1), (4,)), ((2, 1, 1), (8, 1, 1), (8,))]),
    ("kernel rw(global out int o[n], unsigned n) { shared int s[bdim.x]; unsigned t = tid.x; s[t] = t; sync; s[t] = s[t + 1]; sync; o[t] = s[t]; }",
     [((1, 1, 1), (8, 1, 1), (8,)), ((3, 1, 1), (5, 1, 1), (15,))]),
    ("kernel xb(global out int o[4]) { if (tid.x == 0) o[0] = bid.x + 10; if (tid.x == 1) o[1] = o[2]; }",
     [((3, 1, 1), (2, 1, 1), ()), ((1, 1, 1), (2, 1, 1), ())]),
    ("kernel un(global out int o[n], unsigned n) { shared int s[bdim.x]; o[tid.x] = s[tid.x]; }",
     [((2, 1, 1), (4, 1, 1), (8,))]),
    ("kernel lim(global out int o[64]) { for (int i = 0; i < 40; i++) o[i] = i; }", [((1, 1, 1), (1, 1, 1), ())]),
    ("kernel ex(global out int o[4]) { if (tid.x == 0) return; sync; o[tid.x] = 1; }", [((1, 1, 1), (4, 1, 1), ())]),
    ("kernel allx(global out int o[4]) { if (tid.x < 100) return; sync; o[tid.x] = 1; }", [((2, 1, 1), (4, 1, 1), ())]),
    ("kernel sc(global out int o[8], global in int a[4]) { unsigned t = tid.x; int x = (t < 4) && (a[t] != 0);"
     " int y = (t >= 4) || (a[t] == 0); o[t] = (t < 4) ? a[t] : x + y; }", [((1, 1, 1), (8, 1, 1), ())]),
    ("kernel lp(global out int o[8], global in int a[8]) { int s = 0; for (int d = 0; d < a[tid.x] % 7; d++) {"
     " if (d == 2) continue; if (d == 5) break; s += d; } int w = 0; while (w < 7) w += 3; o[tid.x] = s + w; }",
     [((1, 1, 1), (8, 1, 1), ())]),
    ("kernel pa(global out int o[8]) { int a[3]; a[tid.x % 4] = tid.x; o[tid.x] = a[0] + a[1] * 10 + a[(tid.x + 1) % 4]; }",
     [((1, 1, 1), (8, 1, 1), ())]),
    ("kernel fuel(global out int o[2]) { int i = 0; while (tid.x == 0) { i++; } o[tid.x] = i; }",
     [((1, 1, 1), (2, 1, 1), ())]),
    ("kernel ufuel(global out int o[2]) { int i = 0; while (1) { i++; } o[tid.x] = i; }", [((1, 1, 1), (2, 1, 1), ())]),
    ("kernel mix(global inout int a[n], unsigned n) { shared int s[bdim.x]; s[tid.x] = a[tid.x] % 5; sync;"
     " if (s[tid.x] > 2) { a[tid.x] = s[(tid.x + 1) % bdim.x]; } else { s[tid.x] = a[(tid.x * 7) % n] / (s[tid.x] - 1); }"
     " sync; a[tid.x] = a[tid.x] + s[bdim.x - 1 - tid.x]; }",
     [((1, 1, 1), (16, 1, 1), (16,)), ((1, 1, 1), (40, 1, 1), (40,)), ((3, 1, 1), (33, 1, 1), (99,))]),
]


@pytest.mark.parametrize("idx", range(len(FIXTURES)))
def test_fixtures_races_mode(env, oracle, idx):
    text, ls = FIXTURES[idx]
    ref, recs, summ, _ = run_pair(env, oracle, text, None, ls, mode=1, n_seeds=3)
    assert_same(ref, recs, summ)


@pytest.mark.parametrize("bits", [8, 12, 16])
def test_bitwidths(env, oracle, W, bits):
    ls = W.c1_launches()[:150:3]
    ref, recs, summ, _ = run_pair(env, oracle, W.subject("naive_transpose"), W.subject("optimized_transpose"), ls,
                                  n_seeds=2, bits=bits)
    assert_same(ref, recs, summ)
    text, fl = FIXTURES[-1]
    ref, recs, summ, _ = run_pair(env, oracle, text, None, fl, mode=1, n_seeds=2, bits=bits)
    assert_same(ref, recs, summ)


def test_half_warp_bank_model(env, oracle, W):
    ls = [W.scan_launch("prescan", 256, 64), W.scan_launch("prescan", 64, 16)]
    ref, recs, summ, stats = run_pair(env, oracle, W.subject("prescan"), None, ls, mode=2, max_sites=48, n_seeds=1,
                                      bank_model=1)
    assert_same(ref, recs, summ)
    assert (stats == ref["site_stats"]).all()
