"""Run-time barrier divergence (X18; PAPER.md L150-L152 barrier intervals, GKLEE's
deadlock check L55) on the GPU against the oracle, bit-exact: kernels with a `sync` under
thread-dependent control are compiled with per-thread branches and per-thread resume
points; at every round end the live threads' barrier sites are compared and two or more
distinct sites give one BARRIER_DIV event (lowest site, next site, the lowest thread at
each).  Each thread then resumes after its own barrier."""
import pytest

from test_gpu_parity import assert_same, env, run_pair  # noqa: F401  (env: fixture)

pytestmark = pytest.mark.gpu


def L(bdim, gdim=(1, 1, 1), scalars=()):
    b = tuple(bdim) + (1,) * (3 - len(bdim))
    g = tuple(gdim) + (1,) * (3 - len(gdim))
    return (g, b, tuple(scalars))


DIV2 = """
kernel bd(global out int o[n], unsigned n) {
  unsigned g = bid.x * bdim.x + tid.x;
  if (tid.x == 0) { sync; } else { sync; }
  o[g] = 1;
}
"""
DIV3 = """
kernel d3(global out int o[n], unsigned n) {
  unsigned t = tid.x;
  unsigned g = bid.x * bdim.x + t;
  if (t >= 4) { sync; } else { if (t >= 2) { sync; } else { sync; } }
  o[g] = t;
}
"""
UNIFORM_AT_RUNTIME = """
kernel ok(global out int o[n], unsigned n) {
  unsigned g = bid.x * bdim.x + tid.x;
  if (tid.x < bdim.x) { sync; }
  o[g] = 2;
}
"""
EXIT_THEN_SYNC = """
kernel ex(global out int o[n], unsigned n) {
  unsigned g = bid.x * bdim.x + tid.x;
  if (tid.x % 3 == 1) return;
  sync;
  o[g] = 5;
}
"""
# a loop whose trip count depends on the thread: threads leave the loop's barrier at
# different rounds and meet the tail barrier early (divergence in several rounds)
LOOPDIV = """
kernel ld(global out int o[n], global in int a[n], unsigned n) {
  shared int s[bdim.x];
  unsigned t = tid.x;
  unsigned g = bid.x * bdim.x + t;
  s[t] = a[g];
  for (unsigned k = 0; k < t % 4; k++) { s[t] = s[t] + 1; sync; }
  sync;
  o[g] = s[t];
}
"""
# data-dependent barrier (guard reads the input): divergence only for some seeds
DATADIV = """
kernel dd(global out int o[n], global in int a[n], unsigned n) {
  unsigned g = bid.x * bdim.x + tid.x;
  int x = a[g];
  if ((x & 7) == 0) { sync; }
  o[g] = x + 1;
}
"""


def _launches(T, G=(1, 2, 3)):
    return [L((T,), (g,), (T * g,)) for g in G]


@pytest.mark.parametrize("text", [DIV2, DIV3, UNIFORM_AT_RUNTIME, EXIT_THEN_SYNC, LOOPDIV, DATADIV],
                         ids=["two_sites", "three_sites", "uniform_at_runtime", "exit_then_sync", "loop_trip",
                              "data_dependent"])
@pytest.mark.parametrize("T", [1, 6, 32, 48, 256, 1024, 2048])
def test_barrier_divergence_races_mode(env, oracle, text, T):
    ls = _launches(T, G=(1, 3) if T >= 1024 else (1, 2, 3))
    ref, recs, summ, _ = run_pair(env, oracle, text, None, ls, mode=1, n_seeds=5)
    assert_same(ref, recs, summ)


def test_divergence_is_reported_where_expected(env, oracle):
    ls = _launches(8)
    ref, recs, summ, _ = run_pair(env, oracle, DIV3, None, ls, mode=1, n_seeds=2)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][0] == 2 * (1 + 2 + 3)                    # one event per block and seed
    div = [r for r in recs if r[2] == 0]
    assert div and all((r[7], r[12]) == (0, 1) for r in div)          # sites 0 and 1 in every record


def test_divergent_kernel_in_equivalence_check(env, oracle):
    # the divergent kernel against a uniform equivalent: BARRIER_DIV on the source only,
    # outputs equal
    tgt = """
    kernel u(global out int o[n], unsigned n) { unsigned g = bid.x * bdim.x + tid.x; sync; o[g] = 1; }
    """
    ls = _launches(16) + _launches(64)
    ref, recs, summ, _ = run_pair(env, oracle, DIV2, tgt, ls, n_seeds=3)
    assert_same(ref, recs, summ)
    assert summ["per_kind"][5] == 0 and summ["per_kind"][0] > 0


def test_bank_checks_reject_divergent_barriers(env):
    pgvc, torch = env
    k = pgvc.load_ir(DIV2)
    with pytest.raises(pgvc.PgError) as e:
        pgvc.check_banks(k, pgvc.Space(_launches(8)))
    assert e.value.code == pgvc.PG_E_TYPE
