"""Timeline of one check of a bench workload (diagnostics): every evaluation-kernel launch
(kernel, pass, CTA size, start/end ms relative to the check's start) and each kernel's
branch span, from the check graph's event-record nodes (PGVC_TIMELINE=1).
usage: python tools/timeline.py WORKLOAD [seeds] [reps]"""
import os
import sys

os.environ["PGVC_TIMELINE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_lig12_b200 import pgvc, workloads as W  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c2n"
seeds = int(sys.argv[2]) if len(sys.argv) > 2 else 64
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
ws = bench.WORKLOADS[name][3](W, seeds)
st = torch.cuda.Stream()
irs = {}
for w in ws:
    for n in bench.kernel_names(w):
        if n not in irs:
            irs[n] = pgvc.load_ir(W.subject(n))
for w in ws:
    ls, lt = (w.launches[0], None) if hasattr(w, "kernels") else (w.launch_src, w.launch_tgt)
    mode = getattr(w, "input_mode", 0)
    sp = pgvc.Space(ls, lt, n_seeds=seeds if mode != 1 else w.n_seeds, input_mode=mode,
                    input_range=getattr(w, "input_range", 0), checks=w.checks, stream=st.cuda_stream)
    for it in range(reps):
        ref = torch.cuda.Event(enable_timing=True)
        ref.record(st)
        r = bench.run_one(pgvc, irs, w, sp)
        recs, s = r.collect(tuples=False)
        if it == reps - 1:
            print("---- %s: %s" % (name, " ".join(bench.kernel_names(w))), file=sys.stderr)
            r.intervals(ref)
            t = r.timing()
            print("total %.3f ms, K2 sum %.3f ms" % (t["ms_total"], t["ms_eval"]), file=sys.stderr)
