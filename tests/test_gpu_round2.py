"""Round-2 paths of the CUDA path against the oracle, bit for bit:
* store-time claims of the exact protocol (PG_CAS): WW, RW and cross-block
  races on global and shared arrays, in one- and multi-block launches;
* the stamps of single-block launches' global arrays in shared memory (PgArr flags bit 1):
  a read-and-written global array with races, in one block (promoted) and in four (arena);
* the streamed comparison (K3) on array sizes that are not multiples of its 4-cell loads;
* alternating input definitions (RAND32 / RANGE) on one launch list: one plan each.
* thread-private shared stores (PgArr flags bit 2: stores at s[tid.x] in a 1-D block take no
  claim) with RW races, and the same kernels in 2-D blocks, where the stores collide (WW).
The fixtures are small kernels written for these paths (X4 races, X16 records)."""
import pytest

from test_gpu_parity import assert_same, env, run_pair  # noqa: F401  (env: fixture)

pytestmark = pytest.mark.gpu

# a global array read and written by every thread: a RW race between neighbours in round 0
# (thread t reads a[t + 1], which thread t + 1 writes), a WW race on a[0] in round 1, and
# b = a permutation of the result
RACY_GLOBAL = """
kernel g_racy(global inout int a[n], global out int b[n], unsigned n) {
  unsigned t = bid.x * bdim.x + tid.x;
  if (t + 1 < n) a[t] = a[t + 1] + 1;
  sync;
  a[0] = t;
  sync;
  if (t < n) b[t] = a[(t * 7u) % n];
}
"""
# the race-free version: every thread reads its own cell, then writes it after a barrier
CLEAN_GLOBAL = """
kernel g_clean(global inout int a[n], global out int b[n], unsigned n) {
  unsigned t = bid.x * bdim.x + tid.x;
  int x = 0;
  if (t < n) x = a[t];
  sync;
  if (t < n) a[t] = x + 1;
  sync;
  if (t < n) b[t] = a[(t * 7u) % n];
}
"""
# the same pattern on a shared array (claims in s_clm, committed owners in s_own): a load of
# a cell another thread of the round stores to must see the round-start value (X3)
RACY_SHARED = """
kernel s_racy(global in int x[n], global out int y[n], unsigned n) {
  shared int s[bdim.x];
  unsigned t = tid.x;
  unsigned i = bid.x * bdim.x + t;
  s[t] = (i < n) ? x[i] : 0;
  sync;
  if (t + 1 < bdim.x) s[t] = s[t + 1] + s[t];
  if (t == 3u) s[0] = 5;
  sync;
  if (i < n) y[i] = s[(t * 5u) % bdim.x];
}
"""
CLEAN_SHARED = """
kernel s_clean(global in int x[n], global out int y[n], unsigned n) {
  shared int s[bdim.x];
  unsigned t = tid.x;
  unsigned i = bid.x * bdim.x + t;
  s[t] = (i < n) ? x[i] : 0;
  sync;
  int v = s[t];
  if (t + 1 < bdim.x) v = v + s[t + 1];
  sync;
  s[t] = v;
  sync;
  if (i < n) y[i] = s[(t * 5u) % bdim.x];
}
"""


def _launches(W, sizes, blocks):
    out = []
    for n in sizes:
        for g in blocks:
            if n % g == 0:
                out.append(W.Launch((g, 1, 1), (n // g, 1, 1), (n,)))
    return out


@pytest.mark.parametrize("seeds", [1, 5])
def test_global_races_single_and_multi_block(env, oracle, W, seeds):  # noqa: F811
    ls = _launches(W, (1, 2, 7, 32, 100, 1024), (1, 4))
    ref, recs, summ, _ = run_pair(env, oracle, RACY_GLOBAL, CLEAN_GLOBAL, ls, n_seeds=seeds)
    assert_same(ref, recs, summ)
    assert summ["per_kind"] != [0] * 10   # the fixture races and mismatches


def test_global_races_mode(env, oracle, W):  # noqa: F811
    ls = _launches(W, (3, 64, 515, 2048), (1,))
    ref, recs, summ, _ = run_pair(env, oracle, RACY_GLOBAL, None, ls, mode=1, n_seeds=3)
    assert_same(ref, recs, summ)


def test_clean_global_single_block_is_equivalent_to_itself(env, oracle, W):  # noqa: F811
    ls = _launches(W, (5, 256, 4096), (1,))
    ref, recs, summ, _ = run_pair(env, oracle, CLEAN_GLOBAL, CLEAN_GLOBAL, ls, n_seeds=3)
    assert_same(ref, recs, summ)
    assert summ["n_fail"] == 0


@pytest.mark.parametrize("seeds", [1, 9])
def test_shared_races_store_time_claims(env, oracle, W, seeds):  # noqa: F811
    ls = _launches(W, (4, 6, 33, 96, 1024), (1, 2))
    ref, recs, summ, _ = run_pair(env, oracle, RACY_SHARED, CLEAN_SHARED, ls, n_seeds=seeds)
    assert_same(ref, recs, summ)
    assert summ["n_fail"] > 0


def test_compare_ragged_sizes(env, oracle, W):  # noqa: F811
    # output sizes 1, 3, 5, 13, 4099: the 4-cell loads of K3 and their scalar tail
    ls = [W.Launch((1, 1, 1), (n, 1, 1), (n,)) for n in (1, 3, 5, 13)] + \
         [W.Launch((1, 1, 1), (1024, 1, 1), (4099,))]
    ref, recs, summ, _ = run_pair(env, oracle, CLEAN_GLOBAL, RACY_GLOBAL, ls, n_seeds=2)
    assert_same(ref, recs, summ)


def test_alternating_input_definitions(env, oracle, W):  # noqa: F811
    # RAND32 and RANGE(4) on the same launch list, alternating: each its own plan and graph
    w = W.c4("rand", n_seeds=3, max_log_n=6)[0]
    for mode, rng in ((0, 0), (2, 4), (0, 0), (2, 4), (2, 3)):
        ref, recs, summ, _ = run_pair(env, oracle, W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt,
                                      n_seeds=3, input_mode=mode, input_range=rng)
        assert_same(ref, recs, summ)


# thread-private stores (every store at s[t], t = tid.x): RW races between neighbours, a
# thread storing twice in a round, compound stores; in a 2-D block the same stores collide
# (tid.x repeats across tid.y), so the WW races there must still be found (no PG_TP)
TP_RACY = """
kernel tp_racy(global in int x[n], global out int y[n], unsigned n) {
  shared int s[bdim.x];
  unsigned t = tid.x;
  unsigned i = (bid.x * bdim.y + tid.y) * bdim.x + t;
  s[t] = (i < n) ? x[i] : 0;
  sync;
  if (t + 1 < bdim.x) s[t] += s[t + 1];
  s[t] = s[t] + tid.y;
  sync;
  if (i < n) y[i] = s[(t * 3u) % bdim.x];
}
"""
TP_CLEAN = """
kernel tp_clean(global in int x[n], global out int y[n], unsigned n) {
  shared int s[bdim.x];
  unsigned t = tid.x;
  unsigned i = (bid.x * bdim.y + tid.y) * bdim.x + t;
  s[t] = (i < n) ? x[i] : 0;
  sync;
  int v = s[t];
  if (t + 1 < bdim.x) v = v + s[t + 1];
  sync;
  s[t] = v + tid.y;
  sync;
  if (i < n) y[i] = s[(t * 3u) % bdim.x];
}
"""


@pytest.mark.parametrize("seeds", [1, 9])
def test_thread_private_stores(env, oracle, W, seeds):  # noqa: F811
    pgvc, _ = env
    assert pgvc.load_ir(TP_RACY).thread_private() == 0b100 == pgvc.load_ir(TP_CLEAN).thread_private()
    ls = [W.Launch((g, 1, 1), (b, 1, 1), (g * b,)) for b in (1, 2, 5, 32, 64, 256, 1024) for g in (1, 3)]
    ref, recs, summ, _ = run_pair(env, oracle, TP_RACY, TP_CLEAN, ls, n_seeds=seeds)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][3] > 0      # RW races found (X16 kind order: ..., RACE_RW)


def test_thread_private_stores_in_2d_blocks_still_race(env, oracle, W):  # noqa: F811
    ls = [W.Launch((g, 1, 1), (bx, by, 1), (g * bx * by,)) for (bx, by) in ((2, 2), (4, 8), (32, 4), (1, 3))
          for g in (1, 2)]
    ref, recs, summ, _ = run_pair(env, oracle, TP_RACY, TP_CLEAN, ls, n_seeds=3)
    assert_same(ref, recs, summ)
    ref, recs, summ, _ = run_pair(env, oracle, TP_CLEAN, None, ls, mode=1, n_seeds=3)
    assert_same(ref, recs, summ)
    assert summ["n_fail"] > 0           # s[tid.x] from several tid.y: WW


@pytest.mark.parametrize("bits", [8, 12])
def test_narrow_widths_keep_xb_and_ww(env, oracle, W, bits):  # noqa: F811
    # w-bit index arithmetic (X23): at 8 bits tid.x and bid.x wrap at 256, so blocks of 512
    # threads store sdata[tid] to one cell twice (WW) and grids of 512 blocks store
    # g_odata[bid.x] to one cell twice (XB): neither the thread-private nor the
    # block-private shortcut may apply there
    ls, lt = [], []
    for N, B in ((1024, 512), (1024, 2), (8192, 4), (4096, 1024)):
        ls.append(W.reduce_launch("reduce0", N, B))
        lt.append(W.reduce_launch("reduce2", N, B))
    ref, recs, summ, _ = run_pair(env, oracle, W.subject("reduce0"), W.subject("reduce2"), ls, lt, n_seeds=3,
                                  bits=bits)
    assert_same(ref, recs, summ)
    if bits == 8:
        assert summ["per_kind"][2] > 0 and summ["per_kind"][4] > 0    # RACE_WW and RACE_XB
