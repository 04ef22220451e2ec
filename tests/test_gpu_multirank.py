"""The multi-rank path on one GPU (H9): ranks shard the seeds, evaluate on
the device, all_reduce the torch-owned first keys (MIN) and counts (SUM) - gloo here, NCCL on
a multi-GPU box - and collect their own records.  The reduced summary must equal a 1-rank
run and the oracle, and the merged per-rank records the 1-rank record list.  Also runs
bench.py's world > 1 branch with 2 ranks (gloo) against a 1-rank run of the same seeds."""
import json
import os
import socket
import subprocess
import sys

import pytest

from test_gpu_parity import env  # noqa: F401  (fixture)

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    import torch
    import torch.distributed as dist
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_lig12_b200 import distributed as D, pgvc, workloads as W
    w = W.c2_pair("reduce2", "reduce2_obo", n_seeds=6, max_log_n=9, max_log_b=7)
    fk = torch.empty(11, dtype=torch.int64, device="cuda")
    ct = torch.empty(16, dtype=torch.int64, device="cuda")
    sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=6, rank=rank, world=world, checks=w.checks,
                    stream=torch.cuda.current_stream().cuda_stream, first_key=fk, counts=ct)
    run = pgvc.check_equiv(pgvc.load_ir(W.subject(w.src)), pgvc.load_ir(W.subject(w.tgt)), sp)
    D.reduce_summary(fk, ct)              # H9 on the product's own device tensors
    recs, summ = run.collect(cap=1 << 20)  # this rank's own records, the global summary
    out[rank] = (fk.tolist(), ct.tolist(), recs, summ["n_local"], summ["n_records"])
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.timeout(600)
def test_two_ranks_on_one_gpu_match_one_rank_and_oracle(env, oracle, W):  # noqa: F811
    import torch.multiprocessing as mp
    pgvc, torch = env
    from paper_conf_ipps_lig12_b200 import distributed as D
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(2, _port(), out), nprocs=2, join=True)
    w = W.c2_pair("reduce2", "reduce2_obo", n_seeds=6, max_log_n=9, max_log_b=7)
    fk = torch.empty(11, dtype=torch.int64, device="cuda")
    ct = torch.empty(16, dtype=torch.int64, device="cuda")
    sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=6, checks=w.checks,
                    stream=torch.cuda.current_stream().cuda_stream, first_key=fk, counts=ct)
    run = pgvc.check_equiv(pgvc.load_ir(W.subject(w.src)), pgvc.load_ir(W.subject(w.tgt)), sp)
    recs1, _ = run.collect(cap=1 << 20)
    ref = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=6,
                       checks=w.checks, cap=1 << 20)
    for r in range(2):
        keys, counts, _, n_local, n_global = out[r]
        assert keys == fk.tolist() == ref["first_key"]
        assert counts == ct.tolist()
        assert counts[:13] == ref["counts"][:13]
        assert n_global == ref["n_records"] and n_local < n_global    # collect: local records only
    merged = D.merge_records([out[0][2], out[1][2]])
    assert merged == recs1 == ref["records"]


def _bench(world, seeds, port):
    env = dict(os.environ, PGVC_DIST_BACKEND="gloo")
    cmd = [sys.executable, "bench.py", "--gpus", str(world), "--steps", "2", "--warmup", "3", "--seeds", str(seeds),
           "--no-cpu-baseline"]
    if world > 1:
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(world),
               "--master-addr", "127.0.0.1", "--master-port", str(port)] + cmd[1:]
    p = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [l for l in p.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, p.stdout[-2000:]
    return json.loads(lines[0]), p.stderr


@pytest.mark.timeout(2400)
def test_bench_world2_branch_matches_world1(env):  # noqa: F811
    one, _ = _bench(1, 8, 0)
    two, err = _bench(2, 4, _port())
    assert two["n_gpus"] == 2 and one["n_gpus"] == 1
    assert "rank 1/2" in err and "rank 0/2" in err
    # 2 ranks x 4 seeds (seeds r, r+2, ...) = the 1-rank run's 8 seeds: same H9-reduced summary
    assert two["check"] == one["check"]
    assert two["value"] > 0 and two["e2e"]["value"] > 0
    for line in (one, two):
        _bench_contract(line)


def _bench_contract(d):
    # the JSON line's measurement contract: the roofline follows from its own fields
    # (SURVEY.md 8(d)'s per-unit work x the instances of a step / the K2 busy time)
    r = d["roofline"]
    assert r["bound"] == "alu" and r["unit"].startswith("Tops/s")
    per_gpu = d["check"]["instances"] / d["n_gpus"]
    assert abs(r["instances_per_step"] - per_gpu) <= 1e-6 * per_gpu
    achieved = r["algorithmic_ops_per_instance"] * r["instances_per_step"] / (r["k2_busy_ms_per_step"] / 1e3)
    assert abs(r["achieved"] * 1e12 - achieved) <= 1e-6 * achieved
    assert abs(r["frac"] - r["achieved"] / r["peak"]) <= 1e-9
    assert 0 < r["frac"] < 1 and 0 < r["frac_counted_ops"] < r["frac"]
    assert abs(r["frac_of_both_pipes"] - r["achieved"] / r["peak_both_pipes"]) <= 1e-9
    assert r["k2_busy_ms_per_step"] <= d["ms_per_step"] * 1.0001
    assert d["gpu_launches"] > 0 and d["e2e"]["h2d_bytes_per_step"] > 0 and d["e2e"]["d2h_bytes_per_step"] > 0
    assert d["step_ms"]["min"] <= d["step_ms"]["median"] <= d["step_ms"]["max"]
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]


@pytest.mark.timeout(900)
def test_greedy_assignment_subspaces_merge_like_the_whole(env, oracle, W):  # noqa: F811
    """§8(e) greedy (launch, seed) split of C4's exhaustive 0/1 sets (n = 2, 4, 8: 4, 16, 256
    seeds): each rank runs its items as sub-spaces whose key_launch0 / key_seed0 give the
    records their global keys; merged over 3 ranks (MIN keys, SUM counts, records in key
    order) they equal one run per launch - and the oracle's records with the same offsets."""
    pgvc, torch = env
    from paper_conf_ipps_lig12_b200 import distributed as D
    ws = W.c4("bits", max_log_n=3)
    src, tgt = pgvc.load_ir(W.subject(ws[0].src)), pgvc.load_ir(W.subject(ws[0].tgt))
    st = torch.cuda.current_stream().cuda_stream
    costs = [l.bdim[0] * (l.bdim[0].bit_length() ** 2) for w in ws for l in w.launch_src]
    seeds = [w.n_seeds for w in ws]

    def run(l, a, b):
        w = ws[l]
        sp = pgvc.Space(w.launch_src, w.launch_tgt, n_seeds=b - a, seed_base=a, input_mode=1, checks=w.checks,
                        stream=st, key_launch0=l, key_seed0=a)
        recs, summ = pgvc.check_equiv(src, tgt, sp).collect(cap=1 << 20)
        return recs, summ

    whole = [run(l, 0, seeds[l]) for l in range(len(ws))]
    want_recs = sorted((r for recs, _ in whole for r in recs), key=lambda r: r[0])
    want_inst = sum(s["instances"] for _, s in whole)
    want_first = min(s["first_key"] for _, s in whole)
    asg = D.greedy_assignment(costs, seeds, 3, chunk=8)
    got = [run(l, a, b) for items in asg for l, a, b in items]
    assert sorted((r for recs, _ in got for r in recs), key=lambda r: r[0]) == want_recs
    assert sum(s["instances"] for _, s in got) == want_inst
    assert min(s["first_key"] for _, s in got) == want_first
    # the oracle on the same sub-spaces, its keys offset by hand (it has no key offsets)
    for l, w in enumerate(ws):
        ref = oracle.check(W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt, n_seeds=seeds[l],
                           input_mode=1, checks=w.checks, cap=1 << 20)
        mine = [r for r in want_recs if r[3] == l]
        assert [(r[0] + (l << 45),) + tuple(r[1:3]) + (r[3] + l,) + tuple(r[4:]) for r in ref["records"]] == mine
