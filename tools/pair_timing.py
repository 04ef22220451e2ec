"""Per-check K2 / total device time for every pair of a bench workload (diagnostics).
usage: python tools/pair_timing.py WORKLOAD [seeds]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_lig12_b200 import pgvc, workloads as W  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c3"
seeds = int(sys.argv[2]) if len(sys.argv) > 2 else 64
ws = bench.WORKLOADS[name][3](W, seeds)
st = torch.cuda.Stream()
for w in ws:
    src = pgvc.load_ir(W.subject(w.src))
    tgt = pgvc.load_ir(W.subject(w.tgt))
    sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=w.n_seeds, input_mode=w.input_mode,
                    input_range=w.input_range, checks=w.checks, stream=st.cuda_stream)
    for it in range(3):
        r = pgvc.check_equiv(src, tgt, sp)
        recs, s = r.collect(tuples=False)
        t = r.timing()
    print("%-16s vs %-18s launches %4d inst %.3e  K2 %7.2f ms total %7.2f ms  launches %d  -> %.2e inst/s" % (
        w.src, w.tgt, len(w.launch_src), s["instances"], t["ms_eval"], t["ms_total"], t["launches"],
        s["instances"] / (t["ms_total"] / 1e3)))
