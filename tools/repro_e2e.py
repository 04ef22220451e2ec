"""GPU repro of the c2n bench flow: K steps enqueued back to back, then K steps each
synchronised and collected (the e2e phase); reports the first failing call."""
import os, sys, time, traceback
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_lig12_b200 import build, pgvc, workloads as W
build.build()
torch.cuda.set_device(0)
seeds = int(os.environ.get("SEEDS", "64"))
wls = W.c2_all(n_seeds=seeds, max_log_n=int(os.environ.get("LOGN", "16")))
irs = {n: pgvc.load_ir(W.subject(n)) for w in wls for n in w.kernels}
main = torch.cuda.Stream()
side = [torch.cuda.Stream() for _ in wls]
keys = torch.empty(len(wls), 11, dtype=torch.int64, device="cuda")
cnts = torch.empty(len(wls), 16, dtype=torch.int64, device="cuda")
sps = [pgvc.Space(w.launches[0], n_seeds=seeds, checks=w.checks, stream=side[i].cuda_stream, first_key=keys[i],
                  counts=cnts[i]) for i, w in enumerate(wls)]
def step():
    ev = torch.cuda.Event(); ev.record(main)
    runs = []
    for i, (w, sp) in enumerate(zip(wls, sps)):
        side[i].wait_event(ev)
        runs.append(pgvc.check_equiv_n([irs[n] for n in w.kernels], w.launches, sp))
    for s in side: main.wait_stream(s)
    return runs
try:
    for phase in ("burst", "sync"):
        pending = []
        for k in range(int(os.environ.get("K", "10"))):
            runs = step()
            if phase == "sync":
                torch.cuda.synchronize()
                for r in runs: r.collect(cap=1 << 16)
                print(phase, k, "ok", flush=True)
            else:
                pending.append(runs)
        torch.cuda.synchronize()
        for runs in pending:
            for r in runs: r.collect(cap=1 << 16)
        print(phase, "done", flush=True)
        del pending
except Exception:
    traceback.print_exc()
