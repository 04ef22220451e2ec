"""C-ABI library tests that need no GPU: the in-tree libpgvc.so loads, exports
every symbol include/pgvc.h declares, rejects bad input with the right status,
and code-generates + NVRTC-compiles (sm_100a) the evaluation kernel of every
subject in every check variant."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def pgvc():
    from paper_conf_ipps_lig12_b200 import build, pgvc as P
    build.build()
    return P


def declared_functions():
    text = open(os.path.join(ROOT, "include", "pgvc.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(pg_[a-z_]+)\s*\(", text)))


def test_exports_every_declared_symbol(pgvc):
    names = declared_functions()
    assert {"pg_load_ir", "pg_check_equiv", "pg_check_races", "pg_check_banks", "pg_collect_cex"} <= set(names)
    L = ctypes.CDLL(pgvc.LIB_PATH)
    for n in names:
        assert hasattr(L, n), n
    assert set(names) <= set(pgvc.EXPORTS)


def test_struct_sizes_match_header(pgvc):
    assert ctypes.sizeof(pgvc.PgCex) == 64
    assert ctypes.sizeof(pgvc.PgLaunch) == 4 * (3 + 3 + 8 + 1)


@pytest.mark.parametrize("bad,code", [
    ("kernel k(global out int o[4]) { o[0] = x; }", -3),
    ("kernel k(global out int o[4]) { o[0] = 1 }", -2),
])
def test_load_errors(pgvc, bad, code):
    with pytest.raises(pgvc.PgError) as e:
        pgvc.load_ir(bad)
    assert e.value.code == code
    assert re.match(r"\d+:\d+: ", str(e.value).split(": ", 1)[1])


@pytest.mark.parametrize("text,div", [
    ("kernel k(global out int o[4]) { if (tid.x == 0) { sync; } }", 1),
    ("kernel k(global out int o[4]) { for (int i = 0; i < tid.x; i++) { sync; } }", 1),
    ("kernel k(global out int o[4]) { while (o[0] > 0) { sync; } }", 1),
    ("kernel k(global out int o[4]) { for (int i = 0; i < 4; i++) { if (tid.x == i) break; sync; } }", 1),
    ("kernel k(global out int o[4]) { if (bdim.x > 2) { sync; } o[tid.x] = 1; }", 0),
    ("kernel k(global out int o[4]) { for (int i = 0; i < 4; i++) { sync; } }", 0),
])
def test_barriers_under_thread_dependent_control_load(pgvc, text, div):
    """X18 is checked at run time: a `sync` under thread-dependent control (tid or data) loads,
    and is compiled with per-thread branches and resume points (PG_DIVBAR 1); block-uniform
    barriers keep the lock-step code (PG_DIVBAR 0)."""
    src = pgvc.load_ir(text).source()
    assert ("#define PG_DIVBAR %d" % div) in src
    assert "u32 sync_site(u32 k)" in src   # barrier ordinal -> site id of the BARRIER_DIV record


def test_uniform_barriers_accepted(pgvc):
    ok = """kernel k(global out int o[4], int n) {
      shared int s[bdim.x];
      if (tid.x > 2) return;
      for (int i = 0; i < n; i++) { s[tid.x] = i; sync; if (bid.x == 0) { sync; } }
      int m = bdim.x / 2;
      while (m > 0) { sync; m = m >> 1; }
    }"""
    pgvc.load_ir(ok)


SUBJECTS = sorted(f[:-4] for f in os.listdir(os.path.join(ROOT, "subjects")) if f.endswith(".pgk"))


@pytest.mark.parametrize("name", SUBJECTS)
def test_subject_compiles_for_sm100a(pgvc, name):
    from paper_conf_ipps_lig12_b200 import workloads as W
    ir = pgvc.load_ir(W.subject(name))
    fast = 1 << 30   # internal bit: the optimistic pass
    for checks, bits in ((pgvc.CHK_RACE | pgvc.CHK_OOB, 32), (0, 32), (pgvc.CHK_BANK | pgvc.CHK_COALESCE, 32),
                         (pgvc.CHK_RACE | pgvc.CHK_OOB, 8), (pgvc.CHK_RACE | pgvc.CHK_OOB | fast, 32), (fast, 32)):
        ir.compile(bits=bits, checks=checks)


def test_no_cpu_fallback(pgvc):
    # without a GPU the check must fail loudly with PG_E_CUDA, never compute on the host
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_ipps_lig12_b200 import workloads as W
    ir = pgvc.load_ir(W.subject("naive_transpose"))
    with pytest.raises(pgvc.PgError) as e:
        pgvc.check_races(ir, pgvc.Space([((1, 1, 1), (2, 2, 1), (2, 2))]))
    assert e.value.code == pgvc.PG_E_CUDA


# ---------------------------------------------------------------- seed-oblivious analysis (multi-seed lanes)
def test_seed_oblivious_subjects(pgvc, W):
    """Every reduction, scan, transpose, matmul and post-condition kernel takes the same
    accesses for every input; the bitonic networks do not (the compare-exchange stores are
    guarded by the data)."""
    subj = sorted(f[:-4] for f in os.listdir(os.path.join(ROOT, "subjects")) if f.endswith(".pgk"))
    for name in subj:
        ob, nt = pgvc.load_ir(W.subject(name)).seed_oblivious()
        assert ob == (not name.startswith("bitonic")), name
    # reduce3 carries mySum (input-dependent); reduce1 keeps only loop counters and indices
    assert pgvc.load_ir(W.subject("reduce3")).seed_oblivious()[1] >= 1
    assert pgvc.load_ir(W.subject("reduce1")).seed_oblivious()[1] == 0


@pytest.mark.parametrize("body,oblivious", [
    # data only flows into values: oblivious
    ("b[t] = a[t] > 0 ? 1 : 2;", True),
    ("int x = a[t]; int y = x * 3 + t; b[t] = y % 7;", True),
    # an input-dependent address
    ("b[a[t] % n] = 1;", False),
    ("int x = a[t]; b[t] = a[x & 3];", False),
    # an input-dependent guard of a store, of a load, a loop bound
    ("if (a[t] > 0) b[t] = 1;", False),
    ("b[t] = a[t] > 0 ? a[0] : 2;", False),
    ("int k = a[t] & 7; for (int i = 0; i < k; i++) b[t] = i;", False),
    # taint through a variable assigned in a loop
    ("int s = 0; for (int i = 0; i < 4; i++) s = s + a[i]; if (s > 0) b[t] = 1;", False),
])
def test_seed_oblivious_cases(pgvc, body, oblivious):
    text = ("kernel k(global in int a[n], global out int b[n], unsigned n) {\n"
            "  unsigned t = tid.x;\n  %s\n}\n" % body)
    assert pgvc.load_ir(text).seed_oblivious()[0] == oblivious


def test_block_private_subjects(pgvc, W):
    """The SDK reductions write g_odata[bid.x] only (never read): no cell can be shared
    between blocks of a 1-D grid.  The transposes, scans, matmuls and bitonic sorts write
    at thread-dependent indices; the two-pass reduction reads what it writes."""
    subj = sorted(f[:-4] for f in os.listdir(os.path.join(ROOT, "subjects")) if f.endswith(".pgk"))
    private = {n for n in subj if pgvc.load_ir(W.subject(n)).block_private()}
    assert {"reduce0", "reduce1", "reduce2", "reduce2_obo", "reduce3", "reduce4", "reduce5", "reduce6"} <= private
    for n in ("naive_transpose", "optimized_transpose", "prescan", "prescan_padded", "matmul_naive",
              "matmul_tiled", "bitonic_global", "bitonic_shared"):
        assert n not in private, n


@pytest.mark.parametrize("stores,private", [
    ("b[bid.x] = a[tid.x];", True),
    ("if (tid.x == 0) b[(unsigned)bid.x] = 1;", True),
    ("b[bid.x] = 1; b[bid.x] = 2;", True),
    ("b[bid.x + 1] = 1;", False),                  # two blocks can meet on a cell
    ("b[bid.y] = 1;", False),                      # only bid.x is analysed
    ("b[tid.x] = 1;", False),
    ("b[bid.x] = b[bid.x] + 1;", False),           # the output is read
    ("unsigned i = bid.x; b[i] = 1;", False),      # (the index must be bid.x itself)
    ("a[bid.x] = 1;", False),                      # a is read below
])
def test_block_private_cases(pgvc, stores, private):
    text = ("kernel k(global inout int a[n], global out int b[n], unsigned n) {\n"
            "  int x = a[tid.x];\n  %s\n}\n" % stores)
    assert pgvc.load_ir(text).block_private() == private


def test_thread_private_subjects(pgvc, W):
    """sdata[tid] (reduce0, reduce3..6) and sdata[t] with t = tid.x (reduce2 and its off-by-one
    mutant) are thread-private stores; reduce1's sdata[2 s tid], the scans' temp[ai] and the
    transposes' 2-D tile are not."""
    def tp(name):
        return pgvc.load_ir(W.subject(name)).thread_private()
    for n in ("reduce0", "reduce2", "reduce2_obo", "reduce3", "reduce4", "reduce5", "reduce6"):
        assert tp(n) != 0, n
    for n in ("reduce1", "prescan", "prescan_padded", "optimized_transpose", "bitonic_shared", "matmul_tiled"):
        assert tp(n) == 0, n


def test_self_loads_skip_reader_stamps_in_the_optimistic_pass(pgvc, W):
    """reduce2's `sdata[t] += sdata[t + s]`: the load of the thread's own cell (through the
    compound store's index copy, X21) can skip its reader stamp in the optimistic pass when the
    block is 1-D (PgSA::tp); the load of sdata[t + s] keeps it; the exact pass keeps both."""
    k = pgvc.load_ir(W.subject("reduce2"))
    fast = [l for l in k.source(checks=pgvc.CHK_RACE | pgvc.CHK_OOB | (1 << 30)).split("\n") if "pg_ld_sh<" in l]
    exact = [l for l in k.source(checks=pgvc.CHK_RACE | pgvc.CHK_OOB).split("\n") if "pg_ld_sh<" in l]
    assert any("!PG_TP_CONST(2)" in l and ", 3u)" in l for l in fast)      # site 3: sdata[t] (read)
    assert any("<2, true," in l and ", 5u)" in l for l in fast)            # site 5: sdata[t + s]
    assert not any("PG_TP_CONST" in l for l in exact)


@pytest.mark.parametrize("body,private", [
    ("s[tid.x] = a[tid.x];", True),
    ("unsigned t = tid.x; s[t] = 1; s[t] = s[t] + a[t];", True),
    ("unsigned t = tid.x; t = t + 1; s[t] = 1;", False),    # t is not tid.x throughout
    ("s[tid.x + 1] = 1;", False),
    ("s[tid.y] = 1;", False),
    ("if (tid.x == 0) s[0] = 1;", False),
    ("s[(unsigned)tid.x] = 2;", True),
    ("unsigned t = tid.x; s[t] += a[t];", True),            # compound: s[h] with h = t (X21)
    ("unsigned t; s[t] = 1; t = tid.x;", False),            # t is 0 at the store (X21)
    ("unsigned u; unsigned v = u; u = v; s[v] = 1;", False),  # no tid.x at the root
    ("unsigned t = tid.x; if (t < 4u) t = 0; s[t] = 1;", False),
])
def test_thread_private_cases(pgvc, body, private):
    text = ("kernel k(global in int a[n], unsigned n) {\n  shared int s[bdim.x];\n  %s\n}\n" % body)
    assert bool((pgvc.load_ir(text).thread_private() >> 1) & 1) == private    # s is array 1 (a is array 0)


@pytest.mark.parametrize("body,checked,elided", [
    # the back-edge follows the body's last barrier: the first back-edge of its round
    ("for (int i = 0; i < n; i++) { s[tid.x] = i; sync; }", 0, 1),
    ("for (int i = 0; i < n; i++) { for (int j = 0; j < n; j++) s[tid.x] = j; sync; }", 1, 1),
    # a loop between the last barrier and the back-edge can spend the round's fuel first
    ("for (int i = 0; i < n; i++) { sync; for (int j = 0; j < n; j++) s[tid.x] = j; }", 2, 0),
    # `continue` before the barrier reaches the back-edge without it
    ("for (int i = 0; i < n; i++) { if (n > 3) continue; sync; }", 1, 0),
    # no barrier: the loop may iterate within one round
    ("for (int i = 0; i < n; i++) { s[tid.x] = i; }", 1, 0),
])
def test_fuel_check_elision(pgvc, body, checked, elided):
    """X19 fuel: the generated back-edge keeps its limit check unless the back-edge
    is provably the first of its round (codegen first_backedge_of_round)."""
    src = "kernel k(global out int o[4], int n) { shared int s[bdim.x]; %s o[0] = 1; }" % body
    text = pgvc.load_ir(src).source()
    n_bodies = max(1, text.count(" seg(Frame& F") + text.count(" run(Frame& F"))
    assert text.count("++C.ufuel > C.fuel") == checked * n_bodies
    assert text.count("t.fuel += (t.live != 0u); ++C.ufuel;") == elided * n_bodies
