"""pgvc benchmark — VC instances checked per second (BASELINE.json metric).

Workload (N=1 headline, BASELINE.json configs[1] = C2): CUDA SDK reduction variants
reduce0..reduce6 checked pairwise against reduce0 plus the injected off-by-one pair
(reduce2 vs reduce2_obo); B = 2^0..2^10 elements per block, N = B..2^16, 64 seeds
per GPU (RAND32), checks EQUIV|RACE|OOB.  One step = every pair over the whole
space: input generation (K1), both evaluation kernels (K2), comparison (K3),
compaction (K4) and the H9 all_reduce of the first-counterexample key (MIN) and
the counts (SUM).  Multi-GPU: N ranks shard a 64 x N seed space round-robin
(64 seeds per GPU, weak scaling); the only collective is H9.

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
# SURVEY.md §8(d) algorithmic work per instance (thread x round) of a reduction round:
# ~10 integer IR ops + 2 shared loads + 1 shared store = 13 ops.
OPS_PER_INSTANCE = 13
SM_COUNT = 148
ALU_LANES_PER_SM_CLK = 64   # IADD3/LOP3 alu pipe: 4 SMSP x 16 lanes/clk (B300_MICROARCH: rt_SMSP = 2)


WORKLOADS = {
    # name: (description, seeds per GPU, ops per instance, builder(seeds))
    "c2": ("C2: SDK reduce0 vs reduce1..6 + reduce2 vs reduce2_obo, B=2^0..2^10, N=B..2^16, "
           "%d RAND32 seeds per GPU, checks EQUIV|RACE|OOB", 64, 13, lambda W, s: W.c2(n_seeds=s)),
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
WL = "c2"


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


def ncu_profile():
    """The committed ncu summary of the evaluation kernel for this workload ({} if none):
    profiles/r1/k2_traffic.json for C2, profiles/r1/<workload>/k2_traffic.json otherwise."""
    p = os.path.join(ROOT, "profiles", "r1", *(() if WL == "c2" else (WL,)), "k2_traffic.json")
    try:
        with open(p) as f:
            return json.load(f)
    except (OSError, ValueError):
        return {}


# ---------------------------------------------------------------- CPU oracle (reference arm / cpu_baseline)
def _oracle_shard(args):
    rank, world, pts_max_log_n, n_seeds = args
    sys.path.insert(0, ROOT)
    import oracle
    from paper_conf_ipps_lig12_b200 import workloads as W
    inst = 0
    for w in W.c2(n_seeds=n_seeds, max_log_n=pts_max_log_n, max_log_b=10):
        r = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=n_seeds,
                         rank=rank, world=world, checks=w.checks, cap=1 << 16)
        inst += r["counts"][0]
    return inst


def oracle_sample(max_log_n=14, n_seeds=0):
    """The oracle as it stands, one process per host core over seed shards, on the
    C2 pairs restricted to N <= 2^max_log_n and n_seeds seeds (default: one seed per core)."""
    import multiprocessing as mp
    sys.path.insert(0, ROOT)
    import oracle
    oracle.build()
    cores = len(os.sched_getaffinity(0))
    n_seeds = n_seeds or max(4, cores)
    world = min(cores, n_seeds)
    t0 = time.perf_counter()
    with mp.get_context("fork").Pool(world) as pool:
        inst = sum(pool.map(_oracle_shard, [(r, world, max_log_n, n_seeds) for r in range(world)]))
    dt = time.perf_counter() - t0
    sample = ("C2 pairs restricted to N <= 2^%d (B = 2^0..2^10), seeds 0..%d, %d processes"
              % (max_log_n, n_seeds - 1, world))
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
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="pgvc", choices=["pgvc", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--ref-log-n", type=int, default=13, help="reference arm: C2 sample N <= 2^k per step")
    ap.add_argument("--ref-seeds", type=int, default=0, help="0: one seed per host core")
    ap.add_argument("--profile", action="store_true", help="1 warm-up + 1 step, no JSON (for ncu launch lists)")
    ap.add_argument("--diag", action="store_true", help="print per-step enqueue / device / per-check times")
    ap.add_argument("--workload", default="c2", choices=sorted(WORKLOADS),
                    help="c2 (headline, BASELINE configs[1]); others: the remaining configs for reference")
    ap.add_argument("--streams", type=int, default=1,
                    help="streams the independent pairs are spread over (0: one per pair; default 1: one stream, "
                         "DESIGN.md §6 'Concurrent pairs')")
    ap.add_argument("--seeds", type=int, default=0, help="seeds per GPU (default: the workload's)")
    args = ap.parse_args()
    global WL, SEEDS_PER_GPU, OPS_PER_INSTANCE
    WL = args.workload
    SEEDS_PER_GPU = args.seeds or WORKLOADS[WL][1]
    OPS_PER_INSTANCE = WORKLOADS[WL][2]
    if args.impl == "reference":
        run_reference(args)
        return

    import torch
    import torch.distributed as dist
    world, rank, local = dist_env()
    dev = local % max(1, torch.cuda.device_count())   # ranks > #GPUs share devices (tests only)
    torch.cuda.set_device(dev)
    if world > 1:
        backend = os.environ.get("PGVC_DIST_BACKEND", "nccl")   # gloo: several ranks on one GPU (tests)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group(backend)
    from paper_conf_ipps_lig12_b200 import build, distributed, pgvc
    if rank == 0 or world == 1:
        build.build()
    if world > 1:
        dist.barrier()
    wls = c2_pairs()
    irs = {}
    for w in wls:
        for name in (w.src, w.tgt):
            if name not in irs:
                from paper_conf_ipps_lig12_b200 import workloads as W
                irs[name] = pgvc.load_ir(W.subject(name))
    stream = torch.cuda.Stream()
    # the pairs are independent checks: with --streams S > 1 they are spread over S side
    # streams forked from and joined back into `stream` (each pair has its own key/count rows)
    n_side = args.streams if args.streams > 0 else len(wls)
    side = [torch.cuda.Stream() for _ in range(n_side)] if n_side > 1 else [stream]
    pair_keys = torch.empty(len(wls), 11, dtype=torch.int64, device="cuda")
    pair_counts = torch.empty(len(wls), 16, dtype=torch.int64, device="cuda")
    step_keys = torch.empty(11, dtype=torch.int64, device="cuda")
    step_counts = torch.zeros(16, dtype=torch.int64, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")

    def step(keys_out, counts_out):
        """One pass of the whole path over the workload (enqueue only): H1..H8 per pair, H9 at the end."""
        runs = []
        fork = torch.cuda.Event()
        fork.record(stream)
        for i, w in enumerate(wls):
            st = side[i % len(side)]
            if st is not stream and i < len(side):
                st.wait_event(fork)
            # weak scaling: 64 seeds per GPU, seeds j = rank, rank + N, ... of a 64 x N seed space
            ns = SEEDS_PER_GPU * world if w.input_mode != 1 else w.n_seeds   # exhaustive 0/1 sets are fixed
            sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=ns, rank=rank, world=world,
                            input_mode=w.input_mode, input_range=w.input_range,
                            checks=w.checks, stream=st.cuda_stream, first_key=pair_keys[i], counts=pair_counts[i])
            runs.append(pgvc.check_equiv(irs[w.src], irs[w.tgt], sp))
        with torch.cuda.stream(stream):
            for st in side:
                if st is not stream:
                    stream.wait_stream(st)
            torch.amin(pair_keys, 0, out=keys_out)
            torch.sum(pair_counts, 0, out=counts_out)
            distributed.reduce_summary(keys_out, counts_out)   # H9: the only cross-GPU traffic
        return runs

    def collect(runs):
        d2h = 0
        for r in runs:
            recs, s = r.collect(cap=1 << 16, tuples=False)
            d2h += 64 * len(recs) + 8 * (16 + 11)
        return d2h

    # warm-up (also JIT-compiles every evaluation kernel variant, builds the plans, and sizes the
    # memory pool for K steps in flight, the pattern of the device-timed phase)
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

    # ---- device-timed phase: K steps enqueued back to back (L2 flush between steps, outside the
    # timed events); host hiccups are absorbed by the queued work
    keys = [torch.empty(11, dtype=torch.int64, device="cuda") for _ in range(args.steps)]
    cnts = [torch.empty(16, dtype=torch.int64, device="cuda") for _ in range(args.steps)]
    clocks = Clocks(dev)
    gc.disable()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    clocks.wait_first()
    evs, all_runs, host_ms = [], [], []
    for k in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        h0 = time.perf_counter()
        e0.record(stream)
        all_runs.append(step(keys[k], cnts[k]))
        e1.record(stream)
        host_ms.append(1000 * (time.perf_counter() - h0))
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
    launches, h2d, eval_ms = 0, 0, 0.0
    for runs in all_runs:
        for r in runs:
            t = r.timing()
            launches += t["launches"]
            h2d += t["h2d_bytes"]
            eval_ms += t["ms_eval"]
    if args.diag and rank == 0:
        print("device ms per step:", ["%.1f" % x for x in step_ms], file=sys.stderr)
        print("host enqueue ms per step:", ["%.1f" % x for x in host_ms], file=sys.stderr)
        print("step keys/counts:", keys[-1].tolist(), cnts[-1].tolist(), file=sys.stderr)
    del all_runs

    # ---- end-to-end phase: the same steps through the C ABI, host launch lists in, records and
    # counters read back every step (wall clock)
    wall_s, d2h = 0.0, 0
    for k in range(args.steps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        runs = step(keys[k], cnts[k])
        d2h += collect(runs)
        torch.cuda.synchronize()
        wall_s += time.perf_counter() - t0
        del runs
    t = torch.tensor([dev_ms, wall_s], dtype=torch.float64, device="cuda")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    dev_ms, wall_s = float(t[0]), float(t[1])
    value = inst_total / (dev_ms / 1000.0)
    e2e = inst_total / wall_s
    peaks = measured_peaks()
    sm_max = clk.get("sm_max_mhz") or peaks.get("sm_max_mhz", 1965.0)
    alu_peak = SM_COUNT * ALU_LANES_PER_SM_CLK * sm_max * 1e6
    per_gpu_inst = inst_total / world
    # K2 time: with one stream, the sum of the evaluation launches' durations (CUDA events around
    # each); with the pairs on concurrent streams those launches overlap each other and the other
    # kernels, so a launch's duration is no longer the kernel's own - the whole device step time is
    # used instead (a lower bound on K2's achieved rate: it also covers K1/K2b/K3/K4)
    k2_basis = "k2_launches" if len(side) == 1 else "whole_step"
    k2_s = eval_ms / 1000.0 if len(side) == 1 else dev_ms / 1000.0
    achieved_ops = per_gpu_inst * OPS_PER_INSTANCE / k2_s if k2_s else None
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": dev_ms / args.steps, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": workload_desc(), "seeds_per_gpu": SEEDS_PER_GPU, "l2": "flushed between steps",
                   "streams": len(side),
                   "parallelism": "dp%d over seeds" % world},
        "roofline": {"bound": "alu", "achieved": achieved_ops / 1e12 if achieved_ops else None,
                     "peak": alu_peak / 1e12, "unit": "Tops/s (int32, algorithmic IR ops)",
                     "frac": (achieved_ops / alu_peak) if achieved_ops else None,
                     "traffic": ncu_profile().get("bytes_per_launch"),
                     "ncu_issue_active_pct": ncu_profile().get("issue_active_pct_time_weighted"),
                     "kernel": "pgk_eval (K2)", "ops_per_instance": OPS_PER_INSTANCE,
                     "k2_ms_per_step": eval_ms / args.steps, "time_basis": k2_basis, "streams": len(side),
                     "peak_source": "148 SM x 64 int32 lanes/clk x sm_max_mhz (DESIGN.md §6)"},
        "e2e": {"value": e2e, "unit": UNIT, "h2d_bytes_per_step": h2d // args.steps,
                "d2h_bytes_per_step": d2h // args.steps},
        "step_ms": {"median": statistics.median(step_ms), "min": min(step_ms), "max": max(step_ms),
                    "host_enqueue_median": statistics.median(host_ms)},
        "gpu_launches": launches // args.steps * args.steps,
        "clocks": clk,
    }
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        inst, dt, cores, sample = oracle_sample()
        line["cpu_baseline"] = {"value": inst / dt, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample}
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
