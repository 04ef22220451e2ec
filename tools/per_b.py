"""Evaluation-kernel throughput per block size B for one C2 pair (diagnostics)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_lig12_b200 import pgvc, workloads as W  # noqa: E402

src, tgt = (sys.argv[1], sys.argv[2]) if len(sys.argv) > 2 else ("reduce0", "reduce2")
irs = {n: pgvc.load_ir(W.subject(n)) for n in (src, tgt)}
st = torch.cuda.Stream()
LB = [int(x) for x in sys.argv[3].split(",")] if len(sys.argv) > 3 else range(0 if tgt not in W.REDUCE_HALF else 1, 11)
for lb in LB:
    B = 1 << lb
    pts = [(1 << ln, B) for ln in range(lb, 17)]
    ls = [W.reduce_launch(src, N, B) for N, B in pts]
    lt = [W.reduce_launch(tgt, N, B) for N, B in pts]
    sp = pgvc.Space(ls, lt, n_seeds=64, checks=7, stream=st.cuda_stream)
    for it in range(3):
        r = pgvc.check_equiv(irs[src], irs[tgt], sp)
        recs, s = r.collect(tuples=False)
        t = r.timing()
    print("B=%5d  instances %.3e  K2 %.2f ms  total %.2f ms  -> %.2e inst/s (K2)" % (
        B, s["instances"], t["ms_eval"], t["ms_total"], s["instances"] / (t["ms_eval"] / 1e3)))
