"""pgvc benchmark - VC instances checked per second (BASELINE.json metric).

Workload (N=1 headline, BASELINE.json configs[1] = C2, in SURVEY.md §8(d)'s design):
the CUDA SDK reduction variants reduce0..reduce6 and the injected off-by-one reduce2_obo,
each evaluated ONCE per (N, B, seed) and every pair compared (pg_check_equiv_n; 28 pairs,
the 21 of reduce0..6 among them); B = 2^1..2^10 elements per block, N = B..2^16, plus the
B = 1 points as a 4-kernel check (reduce3..6 have no B/2 = 0 thread launch); 64 seeds per
GPU (RAND32), checks EQUIV|RACE|OOB.  One step = both checks over the whole space: input
generation (K1), the evaluation kernels (K2), comparison (K3), compaction (K4), the
device-side merge of the checks' counters (K5) and the H9 all_reduce of the first-
counterexample key (MIN) and the counts (SUM).  `--workload c2` runs C2 as seven pairs
(reduce0 against reduce1..6, reduce2 against reduce2_obo; round 1's design).  Multi-GPU: N
ranks shard a 64 x N seed space round-robin (64 seeds per GPU, weak scaling); the only
collective is H9.

`--impl reference` times the CPU oracle (oracle/, test infrastructure) on the
host cores on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import gc
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "VC instances checked/sec (n x tid x round x seed)"
UNIT = "instances/s"
SEEDS_PER_GPU = 64
# the bounded sample the oracle is timed on (cpu_baseline, --impl reference) and the GPU is
# timed on beside it: the C2 pairs restricted to N <= 2^13, seeds 0..15
SAMPLE_LOG_N = 13
SAMPLE_SEEDS = 16


WORKLOADS = {
    # name: (description, seeds per GPU, (unused), builder(seeds)); the useful work per step is
    # counted by the library itself (PG_CHK_OPCOUNT)
    "c2": ("C2: SDK reduce0 vs reduce1..6 + reduce2 vs reduce2_obo, B=2^0..2^10, N=B..2^16, "
           "%d RAND32 seeds per GPU, checks EQUIV|RACE|OOB", 64, 13, lambda W, s: W.c2(n_seeds=s)),
    "c2n": ("C2, the survey's design: reduce0..reduce6 and reduce2_obo each evaluated once per (N, B, seed), all 28 "
            "pairs compared (pg_check_equiv_n; B = 1 points as a 4-kernel check), B=2^0..2^10, N=B..2^16, "
            "%d RAND32 seeds per GPU, checks EQUIV|RACE|OOB", 64, None, lambda W, s: W.c2_all(n_seeds=s)),
    "c1": ("C1: naive vs shared-memory transpose, bdim in [1,4]^2, up to 16x16 threads (1089 launches), "
           "%d RAND32 seeds per GPU, checks EQUIV|RACE|OOB", 64, 14, lambda W, s: [W.c1(n_seeds=s)]),
    "c3": ("C3: Blelloch scan vs padded scan (LOG_NUM_BANKS 4 and 5) and the dropped-barrier mutant, n <= 2^14, "
           "%d seeds per GPU, checks EQUIV|RACE|OOB|BANK|COALESCE", 64, 15,
           lambda W, s: [W.c3_pair("prescan_padded", 4, s), W.c3_pair("prescan_padded", 5, s),
                         W.c3_pair("prescan_nobarrier", 4, s)]),
    "c4": ("C4: bitonic global vs shared, n = 2^1..2^12, RAND32 + RANGE(4) x %d seeds per GPU + exhaustive 0/1 for "
           "n <= 16", 64, 11, lambda W, s: W.c4("rand", s) + W.c4("range", s) + W.c4("bits")),
    "c5t": ("C5 transpose: naive vs 32x32 tiled transpose, N = 32..1024, %d seeds per GPU", 1250, 14,
            lambda W, s: [W.c5_transpose(n_seeds=s)]),
    # matmul, K = 64: naive ~10 ops/k x 64 + 10 = 650 per thread in 1 round; tiled 2 load rounds (~14)
    # + 2 compute rounds (~10 ops/k x 32) + a store round (~10) = ~678 over 5 rounds: (650 + 678) / 6
    "c5m": ("C5 matmul: naive vs 32x32 tiled, N = 32..1024, K = 64, %d seeds per GPU", 1250, (650 + 678) // 6,
            lambda W, s: [W.c5_matmul(n_seeds=s)]),
}
WL = "c2n"

# SURVEY.md §8(d) "Algorithmic work per instance": IR integer ops per (thread, round) counted
# from the paper's code - the per-unit figure the roofline's `achieved` is built on (reduction
# round ~10; transposes 13 / 14; scan round 13-17; bitonic round 10-11; matmul: naive
# 10 ops/k x K + 10 in 1 round, tiled 2 x 14 + 2 x 10 ops/k x 32 + 10 over 5 rounds, K = 64)
SURVEY_OPS = {"c2": 10.0, "c2n": 10.0, "c1": 13.5, "c5t": 13.5, "c3": 15.0, "c4": 10.5,
              "c5m": (10 * 64 + 10 + 2 * 14 + 2 * 10 * 32 + 10) / 6.0}


def workload_desc():
    return WORKLOADS[WL][0] % SEEDS_PER_GPU


def c2_pairs():
    from paper_conf_ipps_lig12_b200 import workloads as W
    return WORKLOADS[WL][3](W, SEEDS_PER_GPU)


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.thread = None

    def start(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + q,
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 7:
                self.rows.append(parts)

    def wait_first(self, timeout=5.0):
        """Block until nvidia-smi delivers its first sample (its start-up takes longer than a
        short timed region), so every later sample falls inside the region."""
        t0 = time.time()
        while self.proc is not None and not self.rows and time.time() - t0 < timeout:
            time.sleep(0.01)
        self.skip = len(self.rows)

    def wait_sample(self, timeout=1.0):
        """Block until at least one sample was taken after wait_first (the region's)."""
        t0 = time.time()
        while self.proc is not None and len(self.rows) <= getattr(self, "skip", 0) and time.time() - t0 < timeout:
            time.sleep(0.01)

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)
        rows = self.rows[getattr(self, "skip", 0):]   # samples taken inside the timed region
        sm = [float(r[0]) for r in rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in rows for i in range(4) if r[3 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(rows)}


def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return json.load(f)
    except OSError:
        return {}


# ---------------------------------------------------------------- CPU oracle (reference arm / cpu_baseline)
def sample_workloads(max_log_n, n_seeds):
    """The bounded sample of the headline workload (C2 restricted to N <= 2^max_log_n)."""
    from paper_conf_ipps_lig12_b200 import workloads as W
    if WL == "c2n":
        return W.c2_all(n_seeds=n_seeds, max_log_n=max_log_n, max_log_b=10)
    return W.c2(n_seeds=n_seeds, max_log_n=max_log_n, max_log_b=10)


def _oracle_shard(args):
    rank, world, pts_max_log_n, n_seeds, wl = args
    global WL
    WL = wl
    sys.path.insert(0, ROOT)
    import oracle
    from paper_conf_ipps_lig12_b200 import workloads as W
    inst = 0
    for w in sample_workloads(pts_max_log_n, n_seeds):
        if hasattr(w, "kernels"):
            r = oracle.check_n([W.subject(n) for n in w.kernels], w.launches, n_seeds=n_seeds, rank=rank,
                               world=world, checks=w.checks, cap=1 << 16)
        else:
            r = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=n_seeds,
                             rank=rank, world=world, checks=w.checks, cap=1 << 16)
        inst += r["counts"][0]
    return inst


def oracle_sample(max_log_n=SAMPLE_LOG_N, n_seeds=SAMPLE_SEEDS):
    """The oracle as it stands, one process per host core over seed shards, on the
    C2 pairs restricted to N <= 2^max_log_n and seeds 0..n_seeds-1."""
    import multiprocessing as mp
    sys.path.insert(0, ROOT)
    import oracle
    oracle.build()
    cores = len(os.sched_getaffinity(0))
    n_seeds = n_seeds or max(4, cores)
    world = min(cores, n_seeds)
    t0 = time.perf_counter()
    with mp.get_context("fork").Pool(world) as pool:
        inst = sum(pool.map(_oracle_shard, [(r, world, max_log_n, n_seeds, WL) for r in range(world)]))
    dt = time.perf_counter() - t0
    sample = ("%s restricted to N <= 2^%d (B = 2^0..2^10), seeds 0..%d, %d processes"
              % ("C2 (all kernels once, all pairs)" if WL == "c2n" else "C2 pairs", max_log_n, n_seeds - 1, world))
    return inst, dt, world, sample


def run_reference(args):
    world, rank, _ = dist_env()
    if rank != 0:
        return
    inst_total, t_total = 0, 0.0
    for _ in range(args.warmup):
        oracle_sample(max_log_n=args.ref_log_n, n_seeds=args.ref_seeds)
    for _ in range(args.steps):
        inst, dt, cores, sample = oracle_sample(max_log_n=args.ref_log_n, n_seeds=args.ref_seeds)
        inst_total += inst
        t_total += dt
    v = inst_total / t_total
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * t_total / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": workload_desc(), "sample": sample},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- GPU arm
def kernel_names(w):
    return list(w.kernels) if hasattr(w, "kernels") else [w.src, w.tgt]


def run_one(pgvc, irs, w, sp):
    """One check of the workload: a pair (pg_check_equiv) or an N-kernel check."""
    if hasattr(w, "kernels"):
        return pgvc.check_equiv_n([irs[n] for n in w.kernels], w.launches, sp)
    return pgvc.check_equiv(irs[w.src], irs[w.tgt], sp)


def k2_busy(runs, ref_ev):
    """(union, sum) in ms of the evaluation-kernel launch intervals of one step's runs,
    relative to the step's start event (launches of a pair's two kernels and of concurrent
    pairs overlap: the union is K2's busy time)."""
    iv = []
    for r in runs:
        iv.extend(r.intervals(ref_ev))
    tot = sum(b - a for a, b in iv)
    iv.sort()
    union, cur_a, cur_b = 0.0, None, None
    for a, b in iv:
        if cur_b is None or a > cur_b:
            if cur_b is not None:
                union += cur_b - cur_a
            cur_a, cur_b = a, b
        else:
            cur_b = max(cur_b, b)
    if cur_b is not None:
        union += cur_b - cur_a
    return union, tot


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="pgvc", choices=["pgvc", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--ref-log-n", type=int, default=SAMPLE_LOG_N, help="oracle sample: C2 with N <= 2^k")
    ap.add_argument("--ref-seeds", type=int, default=SAMPLE_SEEDS, help="oracle sample: seeds 0..k-1")
    ap.add_argument("--profile", action="store_true", help="1 warm-up + 1 step, no JSON (for ncu launch lists)")
    ap.add_argument("--diag", action="store_true", help="print per-step enqueue / device / per-check times")
    ap.add_argument("--workload", default="c2n", choices=sorted(WORKLOADS),
                    help="c2n (headline, BASELINE configs[1] in the survey's design); c2: the same space as seven "
                         "pairs; others: the remaining configs")
    ap.add_argument("--streams", type=int, default=0,
                    help="streams the independent pairs are spread over (default 0: one per pair; 1: one stream)")
    ap.add_argument("--seeds", type=int, default=0, help="seeds per GPU (default: the workload's)")
    args = ap.parse_args()
    global WL, SEEDS_PER_GPU
    WL = args.workload
    SEEDS_PER_GPU = args.seeds or WORKLOADS[WL][1]
    if args.impl == "reference":
        run_reference(args)
        return

    import torch
    import torch.distributed as dist
    world, rank, local = dist_env()
    dev = local % max(1, torch.cuda.device_count())   # ranks > #GPUs share devices (tests only)
    torch.cuda.set_device(dev)
    backend = None
    if world > 1:
        backend = os.environ.get("PGVC_DIST_BACKEND", "nccl")   # gloo: several ranks on one GPU (tests)
        if backend == "nccl":
            os.environ.setdefault("NCCL_DEBUG", "INFO")          # communicator init lines (ranks / nranks)
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group(backend)
        print("[pgvc] rank %d/%d on cuda:%d, %s process group initialised" % (rank, world, dev, backend),
              file=sys.stderr, flush=True)
    from paper_conf_ipps_lig12_b200 import build, distributed, pgvc
    if rank == 0 or world == 1:
        build.build()
    if world > 1:
        dist.barrier()
    wls = c2_pairs()
    irs = {}
    from paper_conf_ipps_lig12_b200 import workloads as W
    for w in wls:
        for name in kernel_names(w):
            if name not in irs:
                irs[name] = pgvc.load_ir(W.subject(name))
    stream = torch.cuda.Stream()
    # the pairs are independent checks: spread over S side streams forked from and joined
    # back into `stream` (default: one per pair); each pair has its own key/count rows
    n_side = args.streams if args.streams > 0 else len(wls)
    side = [torch.cuda.Stream() for _ in range(n_side)] if n_side > 1 else [stream]
    pair_keys = torch.empty(len(wls), 11, dtype=torch.int64, device="cuda")
    pair_counts = torch.empty(len(wls), 16, dtype=torch.int64, device="cuda")
    step_keys = torch.empty(11, dtype=torch.int64, device="cuda")
    step_counts = torch.zeros(16, dtype=torch.int64, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")

    def spaces(extra_checks=0, ns_fn=None):
        out = []
        for i, w in enumerate(wls):
            # weak scaling: 64 seeds per GPU, seeds j = rank, rank + N, ... of a 64 x N seed space
            mode = getattr(w, "input_mode", 0)
            ns = SEEDS_PER_GPU * world if mode != 1 else w.n_seeds   # exhaustive 0/1 sets are fixed
            ls, lt = (w.launches[0], None) if hasattr(w, "kernels") else (w.launch_src, w.launch_tgt)
            out.append(pgvc.Space(ls, lt, n_seeds=ns, rank=rank, world=world,
                                  input_mode=mode, input_range=getattr(w, "input_range", 0),
                                  checks=w.checks | extra_checks, stream=side[i % len(side)].cuda_stream,
                                  first_key=pair_keys[i], counts=pair_counts[i]))
        return out
    sps = spaces()

    def step(keys_out, counts_out, sp_list=None):
        """One pass of the whole path over the workload (enqueue only): H1..H8 per pair, the
        pairs' counters merged on the device (K5), H9 across ranks at the end."""
        runs = []
        fork = torch.cuda.Event()
        fork.record(stream)
        for i, (w, sp) in enumerate(zip(wls, sp_list or sps)):
            st = side[i % len(side)]
            if st is not stream and i < len(side):
                st.wait_event(fork)
            runs.append(run_one(pgvc, irs, w, sp))
        for st in side:
            if st is not stream:
                stream.wait_stream(st)
        pgvc.merge_counters(pair_keys, pair_counts, keys_out, counts_out, stream.cuda_stream)
        with torch.cuda.stream(stream):
            distributed.reduce_summary(keys_out, counts_out)   # H9: the only cross-GPU traffic
        return runs

    def collect(runs):
        d2h = 0
        for r in runs:
            recs, s = r.collect(cap=1 << 16, tuples=False)
            d2h += 64 * len(recs) + 8 * (16 + 11)
        return d2h

    # warm-up (also JIT-compiles every evaluation kernel variant, builds the plans and their
    # workspaces, captures the check graphs)
    collect(step(step_keys, step_counts))
    if not args.profile:
        for _ in range(max(1, args.warmup - 1)):
            pending = [step(step_keys, step_counts) for _ in range(args.steps)]
            torch.cuda.synchronize()
            for runs in pending:
                collect(runs)
            del pending
    torch.cuda.synchronize()
    if args.profile:
        torch.cuda.cudart().cudaProfilerStart()
        collect(step(step_keys, step_counts))
        torch.cuda.synchronize()
        torch.cuda.cudart().cudaProfilerStop()
        return

    # ---- measurement-only passes (outside the timed region): the INT32 peak of this device,
    # and the useful work of one step = the IR integer operations the subject kernels execute
    # (PG_CHK_OPCOUNT: each instance once, no re-runs)
    peak = pgvc.measure_int32_peak(stream.cuda_stream)
    ops_runs = step(step_keys, step_counts, spaces(pgvc.CHK_OPCOUNT))
    torch.cuda.synchronize()
    ir_ops = sum(r.collect(cap=1)[1]["ir_ops"] for r in ops_runs)   # this rank's
    del ops_runs

    # ---- device-timed phase: K steps enqueued back to back (L2 flushed before every step,
    # outside its events); each step replays the captured check graphs
    keys = [torch.empty(11, dtype=torch.int64, device="cuda") for _ in range(args.steps)]
    cnts = [torch.empty(16, dtype=torch.int64, device="cuda") for _ in range(args.steps)]
    clocks = Clocks(dev)
    gc.disable()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    clocks.wait_first()
    evs, all_runs = [], []
    for k in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        all_runs.append(step(keys[k], cnts[k]))
        e1.record(stream)
        evs.append((e0, e1))
    clocks.wait_sample(timeout=2.0)   # (the enqueued steps are still running: a sample under load)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    gc.enable()
    step_ms = [e0.elapsed_time(e1) for e0, e1 in evs]
    dev_ms = sum(step_ms)
    inst_total = sum(int(c[0].item()) for c in cnts)      # whole job: counts are all-reduced over ranks
    launches, h2d, k2_union, k2_sum = 0, 0, [], []
    for (e0, _), runs in zip(evs, all_runs):
        u, t = k2_busy(runs, e0)
        k2_union.append(u)
        k2_sum.append(t)
        for r in runs:
            tm = r.timing()
            launches += tm["launches"]
            h2d += tm["h2d_bytes"]
    if args.diag and rank == 0:
        print("device ms per step:", ["%.2f" % x for x in step_ms], file=sys.stderr)
        print("K2 busy (union) ms per step:", ["%.2f" % x for x in k2_union], file=sys.stderr)
        print("step keys/counts:", keys[-1].tolist(), cnts[-1].tolist(), file=sys.stderr)
    del all_runs

    # ---- end-to-end phase: the same steps through the C ABI from an idle device, host launch
    # lists in, records and counters read back every step (wall clock); the enqueue part of
    # each step is the host cost of the path
    wall_s, d2h, enq_ms = 0.0, 0, []
    for k in range(args.steps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        runs = step(keys[k], cnts[k])
        enq_ms.append(1000 * (time.perf_counter() - t0))
        d2h += collect(runs)
        torch.cuda.synchronize()
        wall_s += time.perf_counter() - t0
        del runs
    t = torch.tensor([dev_ms, wall_s, sum(k2_union)], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    dev_ms, wall_s, k2_ms = float(t[0]), float(t[1]), float(t[2])
    value = inst_total / (dev_ms / 1000.0)
    e2e = inst_total / wall_s
    sm_max = clk.get("sm_max_mhz") or measured_peaks().get("sm_max_mhz", 1965.0)
    # roofline (per GPU): algorithmic work of this rank's step = SURVEY.md §8(d)'s IR ops per
    # instance x the instances it checked, over the K2 busy time, against SURVEY.md §8(d)'s
    # denominator, the INT32 ALU-pipe peak (148 SMs x 64 lanes/clk x f: IADD3/LOP3/SHF/ISETP,
    # the pipe the IR's adds, logic, shifts and compares issue to), measured live; beside it
    # the fraction of both integer pipes (alu + fma/IMAD: the hard upper bound) and the IR
    # operations the subject kernels actually executed (PG_CHK_OPCOUNT: idle threads of a
    # reduction round count as instances, X19, but execute only the guard)
    k2_s = k2_ms / 1000.0 / args.steps
    per_gpu_inst = inst_total / world / args.steps
    achieved = SURVEY_OPS[WL] * per_gpu_inst / k2_s if k2_s else None
    counted = ir_ops / k2_s if k2_s else None
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": dev_ms / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": workload_desc(), "seeds_per_gpu": SEEDS_PER_GPU, "l2": "flushed before every step",
                   "streams": len(side), "parallelism": "dp%d over seeds" % world},
        "roofline": {"bound": "alu", "achieved": achieved / 1e12 if achieved else None,
                     "peak": peak["alu"] / 1e12, "unit": "Tops/s (int32 IR operations)",
                     "frac": (achieved / peak["alu"]) if achieved else None, "traffic": None,
                     "kernel": "pgk_eval (K2)",
                     "algorithmic_ops_per_instance": SURVEY_OPS[WL],
                     "algorithmic_basis": "SURVEY.md 8(d) IR int ops per (thread, round) x instances per step",
                     "instances_per_step": per_gpu_inst,
                     "counted_ir_ops_per_step": ir_ops,
                     "counted_ir_ops_per_instance": ir_ops / per_gpu_inst if per_gpu_inst else None,
                     "frac_counted_ops": (counted / peak["alu"]) if counted else None,
                     "k2_busy_ms_per_step": k2_ms / args.steps,
                     "k2_launch_sum_ms_per_step": sum(k2_sum) / args.steps,
                     "k2_share_of_step": k2_ms / dev_ms if dev_ms else None,
                     "peak_source": "measured live: pg_measure_int32_peak, LOP3 chains on the alu pipe "
                                    "(SURVEY.md 8(d): 148 SMs x 64 lanes/clk x f)",
                     "peak_both_pipes": peak["mixed"] / 1e12, "peak_fma_pipe": peak["fma"] / 1e12,
                     "frac_of_both_pipes": (achieved / peak["mixed"]) if achieved else None,
                     "time_basis": "union of K2 launch intervals (CUDA events in the check graphs)"},
        "e2e": {"value": e2e, "unit": UNIT, "h2d_bytes_per_step": h2d // args.steps,
                "d2h_bytes_per_step": d2h // args.steps},
        "step_ms": {"median": statistics.median(step_ms), "min": min(step_ms), "max": max(step_ms),
                    "host_enqueue_median": statistics.median(enq_ms)},
        "gpu_launches": launches // args.steps * args.steps,
        "clocks": clk,
        # the last timed step's H9-reduced summary (whole job): first failing key, counts
        "check": {"first_key": int(keys[-1][0].item()), "instances": int(cnts[-1][0].item()),
                  "n_fail": int(cnts[-1][12].item()), "records": int(cnts[-1][11].item()),
                  "per_kind": [int(x) for x in cnts[-1][1:11].tolist()]},
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline and WL in ("c2", "c2n"):
        # (the oracle sample is C2's: the other configs are parity cases, not the headline)
        # like for like: the oracle and the GPU on the same bounded sample (C2 with N <= 2^k, seeds
        # 0..S-1), then the oracle's number as the CPU baseline
        inst, dt, cores, sample = oracle_sample(max_log_n=args.ref_log_n, n_seeds=args.ref_seeds)
        line["cpu_baseline"] = {"value": inst / dt, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample}
        g_inst, g_s = gpu_sample(pgvc, irs, stream, args.ref_log_n, args.ref_seeds)
        line["same_sample"] = {"sample": sample, "oracle": inst / dt, "gpu": g_inst / g_s,
                               "instances_match": g_inst == inst}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def gpu_sample(pgvc, irs, stream, max_log_n, n_seeds, reps=5):
    """The GPU on the oracle's sample (same pairs, launches and seeds; best of reps, device time)."""
    import torch
    wls = sample_workloads(max_log_n, n_seeds)
    fk = torch.empty(len(wls), 11, dtype=torch.int64, device="cuda")
    ct = torch.empty(len(wls), 16, dtype=torch.int64, device="cuda")
    sps = [pgvc.Space(w.launches[0] if hasattr(w, "kernels") else w.launch_src,
                      None if hasattr(w, "kernels") else w.launch_tgt, n_seeds=n_seeds, checks=w.checks,
                      stream=stream.cuda_stream, first_key=fk[i], counts=ct[i]) for i, w in enumerate(wls)]
    best, inst = None, 0
    for _ in range(reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        runs = [run_one(pgvc, irs, w, sp) for w, sp in zip(wls, sps)]
        e1.record(stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        inst = sum(r.collect(cap=1)[1]["instances"] for r in runs)
        best = ms if best is None else min(best, ms)
    return inst, best / 1000.0


if __name__ == "__main__":
    main()
