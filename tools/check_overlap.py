"""Per-check host enqueue and device time of a bench workload, each check alone and all
checks concurrently on their own streams (diagnostics: do a step's checks overlap?).
usage: python tools/check_overlap.py WORKLOAD [reps]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_lig12_b200 import pgvc, workloads as W  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c4"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
ws = bench.WORKLOADS[name][3](W, 64)
irs = {}
for w in ws:
    for n in bench.kernel_names(w):
        if n not in irs:
            irs[n] = pgvc.load_ir(W.subject(n))
streams = [torch.cuda.Stream() for _ in ws]


def space(i, w):
    ls, lt = (w.launches[0], None) if hasattr(w, "kernels") else (w.launch_src, w.launch_tgt)
    mode = getattr(w, "input_mode", 0)
    return pgvc.Space(ls, lt, n_seeds=64 if mode != 1 else w.n_seeds, input_mode=mode,
                      input_range=getattr(w, "input_range", 0), checks=w.checks, stream=streams[i].cuda_stream)


sps = [space(i, w) for i, w in enumerate(ws)]
for it in range(reps):
    alone = []
    for i, w in enumerate(ws):   # each check alone
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = bench.run_one(pgvc, irs, w, sps[i])
        h = time.perf_counter() - t0
        torch.cuda.synchronize()
        d = time.perf_counter() - t0
        alone.append((w.name, h, d, r.timing()["launches"]))
        del r
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    runs = [bench.run_one(pgvc, irs, w, sps[i]) for i, w in enumerate(ws)]
    h = time.perf_counter() - t0
    torch.cuda.synchronize()
    d = time.perf_counter() - t0
    if it == reps - 1:
        for n, hh, dd, nl in alone:
            print("%-20s alone: host %6.2f ms, wall %6.2f ms, launches %d" % (n, 1e3 * hh, 1e3 * dd, nl))
        print("sum alone wall %.2f ms; all concurrently: host %.2f ms, wall %.2f ms" %
              (1e3 * sum(a[2] for a in alone), 1e3 * h, 1e3 * d))
