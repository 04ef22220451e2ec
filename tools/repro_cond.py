"""Small GPU repro: one reduced C2 check (graph capture with conditional re-run nodes)."""
import os, sys, traceback
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_lig12_b200 import build, pgvc, workloads as W
build.build()
torch.cuda.set_device(0)
w = W.c2_pair(sys.argv[1] if len(sys.argv) > 1 else "reduce2", sys.argv[2] if len(sys.argv) > 2 else "reduce2_obo",
              n_seeds=3, max_log_n=6, max_log_b=4)
s, t = pgvc.load_ir(W.subject(w.src)), pgvc.load_ir(W.subject(w.tgt))
for it in range(3):
    try:
        sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=3, checks=w.checks,
                        stream=torch.cuda.current_stream().cuda_stream)
        r = pgvc.check_equiv(s, t, sp)
        recs, summ = r.collect()
        print("iter", it, "ok", summ["instances"], len(recs), r.timing())
    except Exception:
        traceback.print_exc()
        break
