"""Pins for multi-kernel sequences (GKLEE's multi-kernel programs,
PAPER.md L62-L63): phases of one side share their global buffers (by name), a kernel
boundary is a grid-wide barrier, and the two sides' final buffers are compared.

What fixes the expected values: the SDK's two-pass reduction (block sums, then one block
over the block sums) computes Σ inputs mod 2^32 (X11, L465) exactly like the one-thread
specification, so the sequence check finds no mismatch - which can only happen if the
second phase reads the first phase's block sums: run alone (PRF contents for g_odata) it
differs on every seed."""
import pytest


def _run(oracle, W, w, **kw):
    return oracle.check_seq([W.subject(n) for n in w.src], [W.subject(n) for n in w.tgt], w.src_launches,
                            w.tgt_launches, cap=1 << 20, **kw)


def test_two_pass_reduction_equals_the_serial_sum(oracle, W):
    w = W.reduce_two_pass(max_log_n=8, max_log_b=4)
    r = _run(oracle, W, w, n_seeds=3)
    assert r["counts"][1 + 5] == 0 and r["first_key"][0] == 2 ** 63 - 1
    # instances: the phases' own counts add up (each phase runs once per (launch, seed))
    per_phase = [oracle.check(W.subject(n), None, ls, mode=1, n_seeds=3)["counts"][0]
                 for n, ls in zip(w.src + w.tgt, w.src_launches + w.tgt_launches)]
    assert r["counts"][0] == sum(per_phase)


def test_second_phase_alone_reads_prf_not_block_sums(oracle, W):
    w = W.reduce_two_pass(max_log_n=6, max_log_b=3)
    r = oracle.check_seq([W.subject("reduce0_pass2")], [W.subject("sum_serial")], [w.src_launches[1]],
                         w.tgt_launches, n_seeds=2, cap=1 << 20)
    n_inst = len(w.src_launches[0]) * 2
    assert r["counts"][12] == n_inst                     # every (launch, seed) mismatches on g_sum[0]
    mm = [x for x in r["records"] if x[2] == 5]
    assert len(mm) == n_inst and all(x[9] == 0 and x[6] == 0xFFFF for x in mm)


def test_buggy_second_phase_is_caught_per_phase(oracle, W):
    # the off-by-one as the first phase: its races / OOB are reported as phase 0 (kernel 0),
    # the outputs still equal the sum (P3 (iv): the mutant sums correctly under X3)
    w = W.reduce_two_pass(max_log_n=6, max_log_b=3, first="reduce2_obo")
    r = _run(oracle, W, w, n_seeds=2)
    assert r["counts"][1 + 5] == 0
    kinds = {(x[5], x[2]) for x in r["records"]}
    assert kinds and all(k == 0 for k, _ in kinds) and {1, 3} <= {kd for _, kd in kinds}


def test_literal_header_sequence_mismatches_first_at_bdim_4(oracle, W):
    # reduce0_lit (X10, wrong sum first at bdim = 4) as the second phase: the sequence differs
    # from the serial sum first where the second phase has 4 threads (M = N / B = 4)
    w = W.reduce_two_pass(max_log_n=7, max_log_b=3)
    lit = W.subject("reduce0_lit").replace("g_idata", "g_odata").replace("g_odata[gdim.x]", "g_sum[gdim.x]")
    lit = lit.replace("g_odata[bid.x] = sdata[0]", "g_sum[bid.x] = sdata[0]").replace("unsigned n)", "unsigned m)")
    lit = lit.replace("< n)", "< m)").replace("g_odata[n]", "g_odata[m]")
    r = oracle.check_seq([W.subject("reduce0"), lit], [W.subject("sum_serial")], w.src_launches, w.tgt_launches,
                         n_seeds=2, cap=1 << 20)
    pts = [(l.scalars[0], l.gdim[0]) for l in w.src_launches[1]]
    first = min(i for i, l in enumerate(w.src_launches[1]) if l.bdim[0] == 4)
    assert r["first_key"][1 + 5] >> 45 == first
