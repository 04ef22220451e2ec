"""Pins for the oracle functions round 1 left unpinned ("Oracle pins").

Every expected value is derived by hand from the definition cited beside it, or from an
independent Python transcription of the published generator - never from the oracle:

  * PG_BANKS_16_HALFWARP, the CC 1.x bank model (X9; motivation L21-L24, L146-L150):
    hand-derived degrees of stride patterns under 16 banks / half-warps vs 32 banks / warps.
  * RANGE(k) inputs (X8): RAND32 % k with RAND32 transcribed here from SplitMix64.
  * multi-block shared POISON tags (X6): POISON(seed, 0x8000 + array, bid << 20 | idx).
  * the BARRIER_DIV record (X17/X18; GKLEE deadlocks L55, barrier intervals L150-L152).
  * the WW record convention (X16; premise "at most one thread writes", L516-L520).
"""
import pytest

M32 = 0xFFFFFFFF
M64 = 0xFFFFFFFFFFFFFFFF


def py_sm64(x):
    """SplitMix64 (Steele, Lea & Flood 2014), transcribed from its definition."""
    x = (x + 0x9E3779B97F4A7C15) & M64
    x = ((x ^ (x >> 30)) * 0xBF58476D1CE4E5B9) & M64
    x = ((x ^ (x >> 27)) * 0x94D049BB133111EB) & M64
    return x ^ (x >> 31)


def py_rand32(seed, tag, idx):
    """X8: RAND32 = low32(sm(sm(seed) ^ (tag << 48) ^ idx))."""
    return py_sm64(py_sm64(seed) ^ (tag << 48) ^ idx) & M32


def one(scalars=(), bdim=(1, 1, 1), gdim=(1, 1, 1)):
    return (gdim, bdim, tuple(scalars))


def test_python_splitmix_matches_published_outputs():
    # the transcription above is itself pinned by the generator's published outputs
    assert py_sm64(0) == 0xE220A8397B1DCDAF and py_sm64(1) == 0x910A2DEC89025CC1


# ------------------------------------------------------------------ X9 bank models
BANKS = """
kernel banks(global out int o[32]) {
  shared int s[1024];
  unsigned t = tid.x;
  int x = s[t];
  x += s[2 * t];
  x += s[16 * t];
  x += s[17 * t];
  x += s[32 * t];
  x += s[(t % 16) + 32 * (t / 16)];
  x += s[t / 2];
  o[t] = x;
}
"""
# Degree = max over banks of the number of DISTINCT words the access group touches
# (same word = broadcast).  32-bank model: bank = word mod 32, group = the 32 lanes of a
# warp.  CC 1.x half-warp model: bank = word mod 16, group = 16 lanes.
#   s[t]                 32: banks t          -> 1        16: banks t mod 16 in a half -> 1
#   s[2t]                32: {0,2,..,62} -> 2 words per even bank -> 2
#                        16: half 0 words 0..30 even -> banks 0,2,..,14 twice -> 2
#   s[16t]               32: banks {0,16}, 16 words each -> 16
#                        16: every word in bank 0 -> 16
#   s[17t]               32: 17t mod 32 distinct (17 odd) -> 1   16: 17t mod 16 = t mod 16 -> 1
#   s[32t]               32: all bank 0 -> 32      16: all bank 0, 16 per half-warp -> 16
#   s[t%16 + 32(t/16)]   32: lanes t and t+16 share bank t%16 with words t, 32+t -> 2
#                        16: each half touches 16 consecutive words -> 1
#   s[t/2]               pairs of lanes read the same word: 16 words in 16 banks -> 1 (both)
DEG32 = [1, 2, 16, 1, 32, 2, 1]
DEG16 = [1, 2, 16, 1, 16, 1, 1]


@pytest.mark.parametrize("model,want", [(0, DEG32), (1, DEG16)])
def test_bank_model_degrees(oracle, model, want):
    r = oracle.check(BANKS, None, [one(bdim=(32, 1, 1))], mode=oracle.MODE_BANKS, checks=oracle.BANK,
                     bank_model=model, max_sites=8)
    st = r["site_stats"][0, 0]
    assert [int(st[s][3]) for s in range(7)] == want          # max degree per site
    assert [int(st[s][1]) for s in range(7)] == [1 if model == 0 else 2] * 7   # warp accesses
    # BANK records (failing in banks mode) at the conflicted sites; val_a = the degree
    bank = [dict(zip(oracle.REC_FIELDS, x)) for x in r["records"] if x[2] == 6]
    # one event per conflicted warp access: model 0 sites 1, 2, 4, 5; model 1 both half-warps of
    # sites 1, 2, 4
    assert len(bank) == 1 and bank[0]["count"] == (4 if model == 0 else 6)
    # the minimum event (round, array, addr, tid_a, tid_b, site, ...): every conflicted site's
    # record names word 0 (lowest word of the lowest most-loaded bank, bank 0) read by thread 0;
    # tid_b = lowest thread reading another word of bank 0: model 0 s[2t] 16, s[16t] 2, s[32t] 1,
    # s[t%16+32(t/16)] 16 -> site 4 (degree 32); model 1 s[2t] 8, s[16t] 1, s[32t] 1 -> the
    # tie at tid_b = 1 goes to the lower site, 2 (degree 16)
    assert (bank[0]["addr"], bank[0]["tid_a"]) == (0, 0)
    assert (bank[0]["site"], bank[0]["tid_b"], bank[0]["val_a"]) == ((4, 1, 32) if model == 0 else (2, 1, 16))


def test_half_warp_groups_are_16_lanes(oracle):
    # 16 threads: one (partial) warp of 16 lanes in the 32-bank model, one half-warp in the
    # 16-bank model.  32 banks: s[2t] touches 16 distinct even banks (1), s[16t] banks {0, 16}
    # with 8 words each (8), s[32t] 16 words of bank 0 (16).  16 banks: s[2t] 2, s[16t] 16,
    # s[32t] 16.  s[t%16 + 32(t/16)] is s[t] here.
    want = {0: [1, 1, 8, 1, 16, 1, 1], 1: [1, 2, 16, 1, 16, 1, 1]}
    for model in (0, 1):
        r = oracle.check(BANKS, None, [one(bdim=(16, 1, 1))], mode=oracle.MODE_BANKS, checks=oracle.BANK,
                         bank_model=model, max_sites=8)
        st = r["site_stats"][0, 0]
        assert [int(st[s][3]) for s in range(7)] == want[model]


# ------------------------------------------------------------------ X8 RANGE(k)
COPY = """
kernel cp(global out int o[n], global in int a[n], unsigned n) { o[tid.x] = a[tid.x]; }
"""


@pytest.mark.parametrize("k", [1, 2, 4, 7, 1000003])
def test_range_inputs_are_rand32_mod_k(oracle, k):
    n = 64
    for seed in (0, 3, 2 ** 33 + 5):
        init, fin, _ = oracle.exec_kernel(COPY, one((n,), bdim=(n, 1, 1)), seed, input_mode=2, input_range=k)
        # gid: sorted union of global names: a -> 0, o -> 1 (X8)
        assert [int(x) for x in init[0]] == [py_rand32(seed, 0, i) % k for i in range(n)]
        assert [int(x) for x in init[1]] == [py_rand32(seed, 1, i) % k for i in range(n)]
        assert [int(x) for x in fin[1]] == [py_rand32(seed, 0, i) % k for i in range(n)]


def test_range_inputs_masked_to_width(oracle):
    # X2: every value is a w-bit pattern - inputs too (RAND32 % k, then masked)
    n = 16
    init, _, _ = oracle.exec_kernel(COPY, one((n,), bdim=(n, 1, 1)), 9, input_mode=2, input_range=1000, bits=8)
    assert [int(x) for x in init[0]] == [(py_rand32(9, 0, i) % 1000) & 0xFF for i in range(n)]


def test_bits01_inputs(oracle):
    n = 40
    seed = 0xA5A5_1234_0F0F
    init, _, _ = oracle.exec_kernel(COPY, one((n,), bdim=(n, 1, 1)), seed, input_mode=1)
    assert [int(x) for x in init[0]] == [(seed >> i) & 1 for i in range(n)]


# ------------------------------------------------------------------ X6 multi-block poison
POISON = """
kernel pz(global out int o[n], unsigned n) {
  shared int s[bdim.x];
  shared int q[bdim.x];
  unsigned g = bid.x * bdim.x + tid.x;
  o[g] = s[tid.x] + q[bdim.x - 1 - tid.x];
}
"""


def test_shared_poison_is_tagged_by_array_and_block(oracle):
    T, G = 4, 3
    for seed in (0, 77):
        _, fin, counts = oracle.exec_kernel(POISON, one((T * G,), bdim=(T, 1, 1), gdim=(G, 1, 1)), seed)
        want = []
        for b in range(G):
            for t in range(T):
                a = py_rand32(seed, 0x8000 + 0, (b << 20) + t)
                c = py_rand32(seed, 0x8000 + 1, (b << 20) + (T - 1 - t))
                want.append((a + c) & M32)
        assert [int(x) for x in fin[0]] == want
        assert counts[1 + 8] == 2 * T * G          # every read is an UNINIT info event


# ------------------------------------------------------------------ X18 BARRIER_DIV record
DIV = """
kernel bd(global out int o[4]) {
  if (tid.x == 0) { sync; } else { sync; }
  o[tid.x] = 1;
}
"""


def test_barrier_divergence_record(oracle):
    r = oracle.check(DIV, None, [one(bdim=(4, 1, 1))], mode=oracle.MODE_RACES, checks=oracle.RACE | oracle.OOB)
    (rec,) = r["records"]
    d = dict(zip(oracle.REC_FIELDS, rec))
    # sites in source order: sync (0), sync (1), o[...] store (2).  Round 0 ends with thread 0
    # at site 0 and threads 1..3 at site 1: record (round 0, no array, addr 0, lowest thread at
    # the lowest site, lowest thread at the next site, site = that lowest site, val_a = the
    # other site), one event.
    assert (d["kind"], d["round"], d["array"], d["addr"]) == (0, 0, 0xFFFFFFFF, 0)
    assert (d["tid_a"], d["tid_b"], d["site"], d["val_a"], d["val_b"], d["count"]) == (0, 1, 0, 1, 0, 1)
    # each thread resumes after its own barrier: the store runs in round 1 for all threads
    assert r["counts"][0] == 4 * 2
    # first failing key: launch 0, seed 0, kernel 0, kind 0 (BARRIER_DIV ranks first), round 0
    assert r["first_key"][0] == 0


def test_runtime_uniform_barrier_under_thread_control_is_not_divergent(oracle):
    k = """
    kernel ok(global out int o[4]) { if (tid.x < bdim.x) { sync; } o[tid.x] = 2; }
    """
    r = oracle.check(k, None, [one(bdim=(4, 1, 1))], mode=oracle.MODE_RACES, checks=oracle.RACE | oracle.OOB)
    assert r["records"] == [] and r["counts"][0] == 8


def test_divergence_with_three_sites_names_the_two_lowest(oracle):
    k = """
    kernel d3(global out int o[6]) {
      unsigned t = tid.x;
      if (t >= 4) { sync; } else { if (t >= 2) { sync; } else { sync; } }
      o[t] = 3;
    }
    """
    r = oracle.check(k, None, [one(bdim=(6, 1, 1))], mode=oracle.MODE_RACES, checks=oracle.RACE | oracle.OOB)
    (rec,) = r["records"]
    d = dict(zip(oracle.REC_FIELDS, rec))
    # sites: sync(t>=4) = 0, sync(t>=2) = 1, sync(else) = 2; waiting: 4,5 at 0; 2,3 at 1; 0,1 at 2
    assert (d["site"], d["val_a"], d["tid_a"], d["tid_b"]) == (0, 1, 4, 2)


# ------------------------------------------------------------------ X16 WW record convention
WW = """
kernel ww(global out int o[4]) {
  shared int s[2];
  s[0] = tid.x + 10;
  if (tid.x >= 2) { s[1] = tid.x + 20; }
  sync;
  o[tid.x] = s[0] + s[1];
}
"""


def test_ww_record_is_the_committed_write_and_the_writer_pair(oracle):
    # X4/X16: a WW race commits the min-tid writer's value (the unique-writer premise of
    # L516-L520 fails; the least writer is the deterministic choice), and its record names
    # (min writer, max writer), the committed write's site and value; the losing value is not
    # part of any later state, so val_b = 0.  One event per raced cell.
    r = oracle.check(WW, None, [one(bdim=(4, 1, 1))], mode=oracle.MODE_RACES, checks=oracle.RACE | oracle.OOB)
    recs = {x[2]: dict(zip(oracle.REC_FIELDS, x)) for x in r["records"]}
    d = recs[2]
    assert d["count"] == 2                        # cells s[0] and s[1]
    # minimum event: cell s[0]: writers 0..3, committed value 0 + 10, store site 0
    assert (d["round"], d["array"], d["addr"], d["tid_a"], d["tid_b"], d["site"], d["val_a"], d["val_b"]) == \
        (0, 0x100, 0, 0, 3, 0, 10, 0)
    _, fin, _ = oracle.exec_kernel(WW, one(bdim=(4, 1, 1)), 0)
    assert [int(x) for x in fin[0]] == [10 + 22] * 4   # s[1] committed by thread 2 (min writer)


# ------------------------------------------------------------------ X19 loop fuel
def test_loop_fuel_limit_record(oracle):
    # X19: at most 2^20 loop back-edges per thread per round; the thread that exceeds it stops
    # (exits) with a LIMIT record (round, no array, addr 0, its gtid, no second thread, no
    # site, val_a = 2 marks the fuel limit; 1 marks the write-log limit)
    k = """
    kernel spin(global out int o[4]) {
      int x = 0;
      if (tid.x >= 1) { while (x >= 0) { x = x + 1; x = x & 0xFFFF; } }
      o[tid.x] = 1;
    }
    """
    r = oracle.check(k, None, [one(bdim=(3, 1, 1))], mode=oracle.MODE_RACES, checks=oracle.RACE | oracle.OOB)
    (rec,) = r["records"]
    d = dict(zip(oracle.REC_FIELDS, rec))
    assert (d["kind"], d["round"], d["array"], d["addr"], d["tid_a"], d["tid_b"], d["site"], d["val_a"]) == \
        (9, 0, 0xFFFFFFFF, 0, 1, 0xFFFFFFFF, 0xFFFFFFFF, 2)
    assert d["count"] == 2                           # threads 1 and 2
    _, fin, counts = oracle.exec_kernel(k, one(bdim=(3, 1, 1)), 0)
    assert int(fin[0][0]) == 1                       # thread 0 finished; 1 and 2 never reached the store
    assert counts[0] == 3


def test_round_limit_record(oracle):
    # X19 / X16: keys keep 16 round bits (0xFFFF marks MISMATCH / XB), so a block runs rounds
    # 0..0xFFFD; threads still live when round 0xFFFE would begin stop with a LIMIT event
    # (round 0xFFFE, their gtid, val_a = 3).  Instances: T x 0xFFFE rounds.
    k = """
    kernel spin_sync(global out int o[4]) { for (unsigned i = 0; i < 70000; i++) { sync; } o[tid.x] = 1; }
    """
    r = oracle.check(k, None, [one(bdim=(2, 1, 1), gdim=(2, 1, 1))], mode=oracle.MODE_RACES,
                     checks=oracle.RACE | oracle.OOB)
    (rec,) = r["records"]
    d = dict(zip(oracle.REC_FIELDS, rec))
    assert (d["kind"], d["round"], d["array"], d["addr"], d["tid_a"], d["tid_b"], d["site"], d["val_a"], d["count"]) == \
        (9, 0xFFFE, 0xFFFFFFFF, 0, 0, 0xFFFFFFFF, 0xFFFFFFFF, 3, 4)
    assert r["counts"][0] == 4 * 0xFFFE
