"""Host enqueue time vs device time of each C2 pair check (diagnostics)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_lig12_b200 import pgvc, workloads as W  # noqa: E402

wls = W.c2(n_seeds=64)
irs = {n: pgvc.load_ir(W.subject(n)) for w in wls for n in (w.src, w.tgt)}
st = torch.cuda.Stream()
for it in range(3):
    tot_host = 0.0
    runs = []
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for w in wls:
        h0 = time.perf_counter()
        sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=64, checks=w.checks, stream=st.cuda_stream)
        r = pgvc.check_equiv(irs[w.src], irs[w.tgt], sp)
        h1 = time.perf_counter()
        runs.append((w.name, r, h1 - h0))
    torch.cuda.synchronize()
    wall = time.perf_counter() - t0
    for name, r, h in runs:
        t = r.timing()
        print("%-28s host %7.1f ms  device total %7.1f ms  K2 %7.1f ms  launches %d" %
              (name, 1e3 * h, t["ms_total"], t["ms_eval"], t["launches"]))
    print("iteration %d wall %.1f ms" % (it, 1e3 * wall), flush=True)
