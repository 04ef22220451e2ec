"""Multi-process path on CPU (gloo, world_size 2): seed sharding + the H9 reduction
(all_reduce MIN of first keys, SUM of counts) reproduce the single-process result.
The oracle supplies per-shard results (no GPU here); the reduction code is the
same `distributed.reduce_summary` bench.py runs over NCCL."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from paper_conf_ipps_lig12_b200 import distributed as D, workloads as W
    w = W.c1(n_seeds=6)
    ls = w.launch_src[::9]
    r = oracle.check(W.subject(w.src), W.subject(w.tgt), ls, ls, n_seeds=6, rank=rank, world=world)
    fk = torch.tensor(r["first_key"], dtype=torch.int64)
    ct = torch.tensor(r["counts"], dtype=torch.int64)
    D.reduce_summary(fk, ct)
    out[rank] = (fk.tolist(), ct.tolist(), r["records"])
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_gloo_world2_matches_single_process(oracle, W):
    from paper_conf_ipps_lig12_b200 import distributed as D
    mgr = mp.Manager()
    out = mgr.dict()
    port = _free_port()
    mp.spawn(_worker, args=(2, port, out), nprocs=2, join=True)
    w = W.c1(n_seeds=6)
    ls = w.launch_src[::9]
    full = oracle.check(W.subject(w.src), W.subject(w.tgt), ls, ls, n_seeds=6)
    for rank in range(2):
        fk, ct, _ = out[rank]
        assert fk == full["first_key"]
        # counts[11] (records) and [12] (failing instances) are per-rank sums too
        assert ct == full["counts"]
    merged = D.merge_records([out[0][2], out[1][2]])
    assert merged == full["records"]
    fw = D.first_witness(full["first_key"][0])
    first_nonsquare = min(i for i, l in enumerate(ls) if l.bdim[0] != l.bdim[1])
    assert fw["launch"] == first_nonsquare


def test_fake_world_shards_union(oracle, W):
    # sharding logic without any process group: shards r = 0..w-1 in one process
    from paper_conf_ipps_lig12_b200 import distributed as D
    w = W.c2_pair("reduce2", "reduce2_obo", n_seeds=5, max_log_n=6, max_log_b=4)
    src, tgt = W.subject(w.src), W.subject(w.tgt)
    full = oracle.check(src, tgt, w.launch_src, w.launch_tgt, n_seeds=5)
    for world in (2, 3, 5):
        parts = [oracle.check(src, tgt, w.launch_src, w.launch_tgt, n_seeds=5, rank=r, world=world)
                 for r in range(world)]
        assert D.merge_records([p["records"] for p in parts]) == full["records"]
        assert min(p["first_key"][0] for p in parts) == full["first_key"][0]
        assert [sum(p["counts"][i] for p in parts) for i in range(16)] == full["counts"]


def test_oracle_check_parallel_equals_serial(oracle, W):
    # the host-parallel oracle (seed shards over processes, merged as H9 merges ranks) used
    # by the full-size GPU parity tests gives exactly the serial oracle's result
    w = W.c2_pair("reduce2", "reduce2_obo", n_seeds=5, max_log_n=7, max_log_b=5)
    args = (W.subject(w.src), W.subject(w.tgt), w.launch_src, w.launch_tgt)
    a = oracle.check(*args, n_seeds=5, checks=w.checks, cap=1 << 20)
    b = oracle.check_parallel(*args, n_seeds=5, checks=w.checks, cap=1 << 20, processes=3)
    assert a["records"] == b["records"] and a["counts"] == b["counts"] and a["first_key"] == b["first_key"]


def test_greedy_assignment_covers_and_balances():
    from paper_conf_ipps_lig12_b200 import distributed as D
    # C4's exhaustive 0/1 sets: n = 2, 4, 8, 16 threads with 2^n seeds, cost ~ n log^2 n
    ns = [2, 4, 8, 16]
    costs = [n * max(1, (n.bit_length() - 1)) ** 2 for n in ns]
    seeds = [1 << n for n in ns]
    for world in (1, 2, 3, 8):
        asg = D.greedy_assignment(costs, seeds, world)
        seen = {}
        for r, items in enumerate(asg):
            for l, a, b in items:
                for s in range(a, b):
                    assert (l, s) not in seen
                    seen[(l, s)] = r
        assert len(seen) == sum(seeds)                       # every (launch, seed) exactly once
        loads = [sum(costs[l] * (b - a) for l, a, b in items) for items in asg]
        chunk = max(1, sum(seeds) // (8 * world))
        biggest = max(costs) * chunk
        assert max(loads) - min(loads) <= biggest           # LPT: within one item of each other
    # round-robin over seeds would leave ranks 4..7 idle on the 4-seed launch; greedy spreads it
    asg = D.greedy_assignment([1.0], [4], 8, chunk=1)
    assert sum(1 for items in asg if items) == 4
