"""Lock-step comparison of aligned loops (X25) on the
oracle.  Pins:
* reduce0 and reduce1 have identical shared state after every round - the body
  correspondence of PAPER.md L839-L845 (writer s = 2k*t): no divergence anywhere;
* reduce0 vs reduce2 (sequential addressing) first differ after round 1 at sdata[0]
  (a0+a1 vs a0+a_{B/2}), hand-derived;
* the literal L825 loop (X10) first differs from reduce0 after round 1 at sdata[0]
  (it adds sdata[2], reduce0 adds sdata[1]) - the round and cell the comparison
  localises, before any output differs;
* rounds >= lock_rounds are not compared."""
import oracle as O


def launches(W, name, pts):
    return [W.reduce_launch(name, N, B) for N, B in pts]


def test_reduce0_reduce1_never_diverge(oracle, W):
    pts = [(B, B) for B in (2, 4, 8, 16, 64)] + [(256, 32)]
    rows = oracle.lockstep(W.subject("reduce0"), W.subject("reduce1"), launches(W, "reduce0", pts),
                           launches(W, "reduce1", pts), n_seeds=3)
    assert rows == []


def test_reduce0_reduce2_first_divergence(oracle, W):
    pts = [(4, 4), (64, 16)]
    rows = oracle.lockstep(W.subject("reduce0"), W.subject("reduce2"), launches(W, "reduce0", pts),
                           launches(W, "reduce2", pts), n_seeds=2)
    assert len(rows) == 4                                  # every instance diverges
    for r in rows:
        d = dict(zip(O.LOCK_FIELDS, r))
        assert (d["block"], d["round"], d["array"], d["addr"]) == (0, 1, 0x100, 0)
        assert d["written_src"] == d["written_tgt"] == 1 and d["val_src"] != d["val_tgt"]


def test_literal_loop_localised(oracle, W):
    pts = [(4, 4), (8, 8)]
    rows = oracle.lockstep(W.subject("reduce0"), W.subject("reduce0_lit"), launches(W, "reduce0", pts),
                           launches(W, "reduce0_lit", pts), n_seeds=1)
    d = [dict(zip(O.LOCK_FIELDS, r)) for r in rows]
    assert [(x["launch"], x["round"], x["addr"]) for x in d] == [(0, 1, 0), (1, 1, 0)]
    # round 0 (the copy into sdata) agrees: no row for round 0 even with lock_rounds = 1
    assert oracle.lockstep(W.subject("reduce0"), W.subject("reduce0_lit"), launches(W, "reduce0", pts),
                           launches(W, "reduce0_lit", pts), lock_rounds=1) == []
