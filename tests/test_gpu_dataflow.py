"""GPU <-> oracle parity of the data-flow relation (H5).

With PG_CHK_DATAFLOW the evaluation kernel records, for every in-bounds
shared/global read, which write supplied the value: the reader's own write of the
current round, the committed write of (w_block, w_round, w_gtid), or the initial
contents.  This is the bounded form of PAPER.md's fresh-writer instantiation
(Fig. 2; ∃-elimination of the writer, L640-L660).  The oracle's rows
come from or_dataflow, which cross-checks each row against literal enumeration of
every candidate writer (VC-literal mode, test_oracle_vcliteral.py).  The sets of
rows must be identical (the order of reads inside a round is not unique)."""
import pytest

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env(oracle, W):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_ipps_lig12_b200 import build, pgvc
    build.build()
    return pgvc, torch


def gpu_rows(env, text, launches, n_seeds, seed_base, bits=32):
    pgvc, torch = env
    k = pgvc.load_ir(text)
    sp = pgvc.Space(launches, n_seeds=n_seeds, seed_base=seed_base, bits=bits,
                    checks=pgvc.CHK_RACE | pgvc.CHK_OOB | pgvc.CHK_DATAFLOW,
                    stream=torch.cuda.current_stream().cuda_stream)
    run = pgvc.check_races(k, sp)
    rows = run.dataflow()
    recs, summ = run.collect()
    return rows, summ


def check_dataflow(env, oracle, text, launches, n_seeds=2, seed_base=7, bits=32):
    rows, summ = gpu_rows(env, text, launches, n_seeds, seed_base, bits)
    total = 0
    for li, l in enumerate(launches):
        for j in range(n_seeds):
            ref = sorted(oracle.dataflow(text, l, seed_base + j, bits=bits))
            sel = rows[(rows[:, 0] == li) & (rows[:, 1] == j)]
            got = sorted(tuple(int(x) for x in r[2:]) for r in sel)
            if got != ref:
                extra = sorted(set(got) - set(ref))[:3]
                missing = sorted(set(ref) - set(got))[:3]
                raise AssertionError("launch %d seed %d: %d gpu rows vs %d oracle rows; gpu-only %s; oracle-only %s"
                                     % (li, j, len(got), len(ref), extra, missing))
            total += len(ref)
    assert len(rows) == total
    return summ


def test_dataflow_transpose(env, oracle, W):
    ls = [W.Launch((2, 2, 1), (4, 4, 1), (8, 8)), W.Launch((3, 2, 1), (4, 4, 1), (10, 7)),
          W.Launch((1, 1, 1), (8, 8, 1), (5, 8))]
    for name in ("naive_transpose", "optimized_transpose", "optimized_transpose_unpadded"):
        check_dataflow(env, oracle, W.subject(name), ls)


@pytest.mark.parametrize("name", ["reduce0", "reduce1", "reduce2", "reduce2_obo", "reduce3", "reduce4",
                                  "reduce5", "reduce6"])
def test_dataflow_reductions(env, oracle, W, name):
    ls = [W.reduce_launch(name, 64, 16), W.reduce_launch(name, 256, 64), W.reduce_launch(name, 32, 32)]
    check_dataflow(env, oracle, W.subject(name), ls)


def test_dataflow_scan_bitonic_matmul(env, oracle, W):
    for name in ("prescan", "prescan_padded", "prescan_nobarrier"):
        check_dataflow(env, oracle, W.subject(name), [W.scan_launch(name, 32, 8), W.scan_launch(name, 64, 16)])
    for name in ("bitonic_global", "bitonic_shared"):
        check_dataflow(env, oracle, W.subject(name), [W.bitonic_launch(name, 16), W.bitonic_launch(name, 32)])
    for name in ("matmul_tiled", "matmul_tiled_nobarrier", "matmul_naive"):
        check_dataflow(env, oracle, W.subject(name), [W.Launch((2, 2, 1), (4, 4, 1), (8, 8, 8))], n_seeds=1)


def test_dataflow_fixtures(env, oracle):
    from test_gpu_parity import FIXTURES
    for text, ls in FIXTURES:
        check_dataflow(env, oracle, text, [tuple(l) for l in ls], n_seeds=2)


def test_dataflow_bits(env, oracle, W):
    for bits in (8, 16):
        check_dataflow(env, oracle, W.subject("reduce1"), [W.reduce_launch("reduce1", 16, 8)], bits=bits)


def test_dataflow_rejected_without_flag(env, W):
    pgvc, torch = env
    k = pgvc.load_ir(W.subject("reduce1"))
    run = pgvc.check_races(k, pgvc.Space([W.reduce_launch("reduce1", 16, 8)],
                                         stream=torch.cuda.current_stream().cuda_stream))
    with pytest.raises(pgvc.PgError):
        run.dataflow()
