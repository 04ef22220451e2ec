"""Minimal failing parameter search.

PUGpara's symmetry-reduction outlook asks for the minimum n at
which a property must be checked.  The bounded analogue: given launches grouped by
an increasing size key n, find the smallest n with a failing instance without
checking every larger n.  Checks run on growing prefixes of the n values (doubling
the number of n values per call), and within one call the first-witness key (X16)
already names the smallest failing launch of that prefix, so the total work is at
most about twice the work of checking up to the witness.

This module is host orchestration only: every check is one call through the C ABI
(`pgvc.check_*`); no evaluation happens here.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Callable, List, Optional, Sequence, Tuple


@dataclass
class Witness:
    n: object                 # the size key of the failing launch
    launch_index: int         # index into the flattened launch list
    launch: object
    summary: dict             # pg_summary of the call that found it
    records: list             # records of the failing launch (canonical order)
    launches_checked: int     # launches checked over all calls
    calls: int


def first_failing(groups: Sequence[Tuple[object, Sequence]], run: Callable[[List, int], Tuple[list, dict]],
                  first_prefix: int = 1) -> Optional[Witness]:
    """groups: [(n, [launch, ...]), ...] in increasing n (the witness order).
    run(launches, offset) checks `launches` (offset = index of its first launch in the
    flattened list) and returns (records, summary) as Run.collect does.
    Returns the minimal failing launch, or None if no launch fails."""
    flat, key_of = [], []
    for n, ls in groups:
        for l in ls:
            flat.append(l)
            key_of.append(n)
    bounds = []                      # end index (exclusive) of each n group in flat
    e = 0
    for _, ls in groups:
        e += len(ls)
        bounds.append(e)
    done_groups, width, checked, calls = 0, max(1, first_prefix), 0, 0
    while done_groups < len(groups):
        lo = bounds[done_groups - 1] if done_groups else 0
        hi_group = min(len(groups), done_groups + width)
        hi = bounds[hi_group - 1]
        recs, summ = run(flat[lo:hi], lo)
        calls += 1
        checked += hi - lo
        if summ["first_launch"] != 0xFFFFFFFF:
            li = lo + summ["first_launch"]
            mine = [r for r in recs if r[3] == summ["first_launch"]]
            return Witness(key_of[li], li, flat[li], summ, mine, checked, calls)
        done_groups = hi_group
        width *= 2
    return None


def equiv_runner(pgvc, src, tgt, n_seeds: int = 8, tgt_of: Optional[Callable] = None, **space_kw):
    """A `run` for first_failing that calls pg_check_equiv (tgt_of maps a source launch to
    the target's, e.g. the B/2-thread reduction variants)."""
    def run(launches, offset):
        lt = [tgt_of(l) for l in launches] if tgt_of else None
        sp = pgvc.Space(list(launches), lt, n_seeds=n_seeds, **space_kw)
        return pgvc.check_equiv(src, tgt, sp).collect()
    return run


def property_runner(pgvc, kernel, post, n_seeds: int = 8, **space_kw):
    """A `run` for first_failing that calls pg_check_property."""
    def run(launches, offset):
        return pgvc.check_property(kernel, post, pgvc.Space(list(launches), None, n_seeds=n_seeds, **space_kw)).collect()
    return run
