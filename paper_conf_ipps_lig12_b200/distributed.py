"""H9 — cross-GPU reduction of one check's summary.

The parameter space shards by seed (rank r takes seeds r, r + world, ...; or, in
weak-scaling runs, its own seed range), so evaluation needs no communication.
Only the first-counterexample keys (int64[11], all_reduce MIN) and the counts
(int64[16], all_reduce SUM) cross the interconnect - NCCL over NVLink on the GPU
box, gloo in the CPU tests.  Records stay on their rank; `merge_records` merges
the per-rank lists on the host (canonical key order is preserved because keys
embed (launch, seed_idx, kernel, kind, round), X16).
"""
from __future__ import annotations

import heapq
from typing import Iterable, List, Sequence

INT64_MAX = 2 ** 63 - 1


def reduce_summary(first_key, counts, group=None):
    """In place: first_key <- MIN over ranks, counts <- SUM over ranks (torch tensors)."""
    import torch.distributed as dist
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(first_key, op=dist.ReduceOp.MIN, group=group)
        dist.all_reduce(counts, op=dist.ReduceOp.SUM, group=group)
    return first_key, counts


def merge_records(per_rank: Sequence[Iterable[tuple]]) -> List[tuple]:
    """Merge per-rank record lists (each already in canonical order) by (key, array, addr, tid_a, tid_b)."""
    def order(r):
        # REC_FIELDS = key, count, kind, launch, seed_idx, kernel, round, site, array, addr, tid_a, tid_b, ...
        return (r[0], r[8], r[9], r[10], r[11])
    return list(heapq.merge(*[list(p) for p in per_rank], key=order))


def first_witness(first_key: int):
    """Decode the first-witness launch / seed index from a key (X16); None if no failure."""
    if first_key >= INT64_MAX:
        return None
    return {"launch": first_key >> 45, "seed_idx": (first_key >> 24) & 0x1FFFFF, "kernel": (first_key >> 20) & 0xF,
            "kind": (first_key >> 16) & 0xF, "round": first_key & 0xFFFF}
