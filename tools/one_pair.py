"""One C2 pair checked `reps` times on the whole C2 space (diagnostics, e.g. under ncu).
usage: python tools/one_pair.py SRC TGT [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_lig12_b200 import pgvc, workloads as W  # noqa: E402

src, tgt = sys.argv[1], sys.argv[2]
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
w = [p for p in W.c2(n_seeds=64) if p.src == src and p.tgt == tgt][0]
irs = pgvc.load_ir(W.subject(src)), pgvc.load_ir(W.subject(tgt))
st = torch.cuda.Stream()
sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=w.n_seeds, checks=w.checks, stream=st.cuda_stream)
for it in range(reps):
    if it == reps - 1:
        torch.cuda.cudart().cudaProfilerStart()
    r = pgvc.check_equiv(irs[0], irs[1], sp)
    recs, s = r.collect(tuples=False)
    t = r.timing()
torch.cuda.cudart().cudaProfilerStop()
print(src, tgt, s["instances"], t)
