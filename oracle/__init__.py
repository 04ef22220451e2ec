"""CPU oracle for pgvc — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this package.  The product path
(paper_conf_ipps_lig12_b200/) never imports it, and it never imports the
product: the two share no code, only the launch lists of
paper_conf_ipps_lig12_b200/workloads.py (input definition).

The oracle itself is oracle/pg_oracle.cpp: a plain sequential tree-walking
interpreter of the kernel IR under PUGpara's barrier-round semantics
(PAPER.md L150-L152, L379-L444, L478-L733), with its own parser and PRF.
Parity status per function is listed in DESIGN.md §"Oracle pins".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "pg_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

EQUIV, RACE, OOB, BANK, COALESCE = 1, 2, 4, 8, 16
MODE_EQUIV, MODE_RACES, MODE_BANKS = 0, 1, 2
KINDS = ["BARRIER_DIV", "OOB", "RACE_WW", "RACE_RW", "RACE_XB", "MISMATCH", "BANK", "UNCOALESCED", "UNINIT", "LIMIT"]


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain g++, no CUDA)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp.%d" % os.getpid()
        subprocess.check_call(["g++", "-std=c++17", "-O2", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


class OrLaunch(ctypes.Structure):
    _fields_ = [("gdim", ctypes.c_uint32 * 3), ("bdim", ctypes.c_uint32 * 3),
                ("scalar", ctypes.c_int32 * 8), ("n_scalar", ctypes.c_uint32)]


class OrRec(ctypes.Structure):
    _fields_ = [("key", ctypes.c_uint64), ("count", ctypes.c_uint64)] + [
        (n, ctypes.c_uint32) for n in ("kind", "launch", "seed_idx", "kernel", "round", "site", "array", "addr",
                                       "tid_a", "tid_b", "val_a", "val_b")]


class OrSpace(ctypes.Structure):
    _fields_ = [("launch_src", ctypes.POINTER(OrLaunch)), ("launch_tgt", ctypes.POINTER(OrLaunch)),
                ("n_launch", ctypes.c_uint32), ("seed_base", ctypes.c_uint64), ("n_seeds", ctypes.c_uint32),
                ("rank", ctypes.c_uint32), ("world", ctypes.c_uint32), ("input_mode", ctypes.c_uint32),
                ("input_range", ctypes.c_uint32), ("bits", ctypes.c_uint32), ("checks", ctypes.c_uint32),
                ("bank_model", ctypes.c_uint32), ("wmax", ctypes.c_uint32), ("mode", ctypes.c_uint32),
                ("vcliteral", ctypes.c_uint32), ("max_sites", ctypes.c_uint32)]


REC_FIELDS = ("key", "count", "kind", "launch", "seed_idx", "kernel", "round", "site", "array", "addr",
              "tid_a", "tid_b", "val_a", "val_b")


def lib():
    global _lib
    with _lock:
        if _lib is None:
            _lib = ctypes.CDLL(build())
            _lib.or_check.restype = ctypes.c_int
            _lib.or_check.argtypes = [ctypes.c_char_p, ctypes.c_char_p, ctypes.POINTER(OrSpace),
                                      ctypes.POINTER(OrRec), ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64),
                                      ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64),
                                      ctypes.POINTER(ctypes.c_uint64)]
            _lib.or_check_n.restype = ctypes.c_int
            _lib.or_check_n.argtypes = [ctypes.POINTER(ctypes.c_char_p), ctypes.c_uint32,
                                        ctypes.POINTER(ctypes.POINTER(OrLaunch)), ctypes.POINTER(OrSpace),
                                        ctypes.POINTER(OrRec), ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64),
                                        ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64),
                                        ctypes.POINTER(ctypes.c_uint64)]
            _lib.or_check_seq.restype = ctypes.c_int
            _lib.or_check_seq.argtypes = [ctypes.POINTER(ctypes.c_char_p), ctypes.c_uint32, ctypes.c_uint32,
                                          ctypes.POINTER(ctypes.POINTER(OrLaunch)), ctypes.POINTER(OrSpace),
                                          ctypes.POINTER(OrRec), ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64),
                                          ctypes.POINTER(ctypes.c_int64), ctypes.POINTER(ctypes.c_int64)]
            _lib.or_exec.restype = ctypes.c_int
            _lib.or_exec.argtypes = [ctypes.c_char_p, ctypes.POINTER(OrLaunch), ctypes.c_uint64, ctypes.c_uint32,
                                     ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                     ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32),
                                     ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint32), ctypes.c_uint32,
                                     ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_int64)]
            _lib.or_dataflow.restype = ctypes.c_int
            _lib.or_dataflow.argtypes = [ctypes.c_char_p, ctypes.POINTER(OrLaunch), ctypes.c_uint64,
                                         ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint32), ctypes.c_uint64,
                                         ctypes.POINTER(ctypes.c_uint64)]
            _lib.or_lockstep.restype = ctypes.c_int
            _lib.or_lockstep.argtypes = [ctypes.c_char_p, ctypes.c_char_p, ctypes.POINTER(OrSpace), ctypes.c_uint32,
                                         ctypes.POINTER(ctypes.c_uint32), ctypes.c_uint64,
                                         ctypes.POINTER(ctypes.c_uint64)]
            _lib.or_last_error.restype = ctypes.c_char_p
            _lib.or_sm64.restype = ctypes.c_uint64
            _lib.or_sm64.argtypes = [ctypes.c_uint64]
            _lib.or_rand32.restype = ctypes.c_uint32
            _lib.or_rand32.argtypes = [ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64]
        return _lib


class OracleError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__("oracle error %d: %s" % (code, msg))
        self.code = code


def _launch(l) -> OrLaunch:
    gdim, bdim, sc = (l.gdim, l.bdim, l.scalars) if hasattr(l, "gdim") else l
    o = OrLaunch()
    for i in range(3):
        o.gdim[i] = gdim[i]
        o.bdim[i] = bdim[i]
    for i, v in enumerate(sc):
        o.scalar[i] = v
    o.n_scalar = len(sc)
    return o


def _launch_array(ls):
    arr = (OrLaunch * max(1, len(ls)))()
    for i, l in enumerate(ls):
        arr[i] = _launch(l)
    return arr


def check(src: str, tgt, launch_src, launch_tgt=None, *, n_seeds=1, seed_base=0, rank=0, world=1,
          input_mode=0, input_range=0, bits=32, checks=EQUIV | RACE | OOB, bank_model=0, wmax=32,
          mode=MODE_EQUIV, vcliteral=False, max_sites=0, cap=1 << 16):
    """Run the oracle over (launches x seeds).  Returns dict with
    records (list of tuples in REC_FIELDS order, canonical key order),
    counts (16 int64), first_key (11 int64), site_stats (ndarray or None)."""
    L = lib()
    ls = _launch_array(launch_src)
    lt = _launch_array(launch_tgt) if launch_tgt is not None else None
    sp = OrSpace()
    sp.launch_src = ctypes.cast(ls, ctypes.POINTER(OrLaunch))
    sp.launch_tgt = ctypes.cast(lt, ctypes.POINTER(OrLaunch)) if lt is not None else None
    sp.n_launch = len(launch_src)
    sp.seed_base = seed_base
    sp.n_seeds = n_seeds
    sp.rank, sp.world = rank, world
    sp.input_mode, sp.input_range, sp.bits = input_mode, input_range, bits
    sp.checks, sp.bank_model, sp.wmax, sp.mode = checks, bank_model, wmax, mode
    sp.vcliteral = 1 if vcliteral else 0
    sp.max_sites = max_sites
    recs = (OrRec * cap)()
    n = ctypes.c_uint64(0)
    counts = (ctypes.c_int64 * 16)()
    first = (ctypes.c_int64 * 11)()
    stats = None
    stats_ptr = None
    if max_sites:
        stats = np.zeros((len(launch_src), 2, max_sites, 8), dtype=np.uint64)
        stats_ptr = stats.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))
    rc = L.or_check(src.encode(), tgt.encode() if tgt else None, ctypes.byref(sp), recs, cap, ctypes.byref(n),
                    counts, first, stats_ptr)
    if rc != 0:
        raise OracleError(rc, L.or_last_error().decode())
    m = min(n.value, cap)
    out = [tuple(getattr(recs[i], f) for f in REC_FIELDS) for i in range(m)]
    return {"records": out, "n_records": n.value, "counts": list(counts), "first_key": list(first),
            "site_stats": stats}


def check_n(texts, launches, *, n_seeds=1, seed_base=0, rank=0, world=1, input_mode=0, input_range=0, bits=32,
            checks=EQUIV | RACE | OOB, wmax=32, cap=1 << 16):
    """N-kernel check (or_check_n): every kernel once per (launch, seed), every pair i < j
    compared, a pair's mismatch in kernel i's MISMATCH slot with site = j.  launches[k] is
    kernel k's launch list.  Same result dict as check()."""
    L = lib()
    nk = len(texts)
    arrs = [_launch_array(ls) for ls in launches]
    ptrs = (ctypes.POINTER(OrLaunch) * nk)(*[ctypes.cast(a, ctypes.POINTER(OrLaunch)) for a in arrs])
    tx = (ctypes.c_char_p * nk)(*[t.encode() for t in texts])
    sp = OrSpace()
    sp.launch_src = ptrs[0]
    sp.launch_tgt = None
    sp.n_launch = len(launches[0])
    sp.seed_base, sp.n_seeds, sp.rank, sp.world = seed_base, n_seeds, rank, world
    sp.input_mode, sp.input_range, sp.bits = input_mode, input_range, bits
    sp.checks, sp.wmax, sp.mode = checks, wmax, MODE_EQUIV
    recs = (OrRec * cap)()
    n = ctypes.c_uint64(0)
    counts = (ctypes.c_int64 * 16)()
    first = (ctypes.c_int64 * 11)()
    rc = L.or_check_n(tx, nk, ptrs, ctypes.byref(sp), recs, cap, ctypes.byref(n), counts, first, None)
    if rc != 0:
        raise OracleError(rc, L.or_last_error().decode())
    m = min(n.value, cap)
    out = [tuple(getattr(recs[i], f) for f in REC_FIELDS) for i in range(m)]
    return {"records": out, "n_records": n.value, "counts": list(counts), "first_key": list(first),
            "site_stats": None}


def check_seq(src_texts, tgt_texts, src_launches, tgt_launches, *, n_seeds=1, seed_base=0, rank=0, world=1,
              input_mode=0, input_range=0, bits=32, checks=EQUIV | RACE | OOB, wmax=32, cap=1 << 16):
    """Multi-kernel sequences (or_check_seq): the source kernels run in order on one set of
    global buffers (matched by name), so do the target kernels; final buffers compared.
    src_launches[i] / tgt_launches[i]: launch list of phase i (same length for all).
    Records: kernel = phase index (source phases first)."""
    L = lib()
    texts = list(src_texts) + list(tgt_texts)
    launches = list(src_launches) + list(tgt_launches)
    nk = len(texts)
    arrs = [_launch_array(ls) for ls in launches]
    ptrs = (ctypes.POINTER(OrLaunch) * nk)(*[ctypes.cast(a, ctypes.POINTER(OrLaunch)) for a in arrs])
    tx = (ctypes.c_char_p * nk)(*[t.encode() for t in texts])
    sp = OrSpace()
    sp.launch_src = ptrs[0]
    sp.launch_tgt = None
    sp.n_launch = len(launches[0])
    sp.seed_base, sp.n_seeds, sp.rank, sp.world = seed_base, n_seeds, rank, world
    sp.input_mode, sp.input_range, sp.bits = input_mode, input_range, bits
    sp.checks, sp.wmax, sp.mode = checks, wmax, MODE_EQUIV
    recs = (OrRec * cap)()
    n = ctypes.c_uint64(0)
    counts = (ctypes.c_int64 * 16)()
    first = (ctypes.c_int64 * 11)()
    rc = L.or_check_seq(tx, nk, len(src_texts), ptrs, ctypes.byref(sp), recs, cap, ctypes.byref(n), counts, first)
    if rc != 0:
        raise OracleError(rc, L.or_last_error().decode())
    m = min(n.value, cap)
    out = [tuple(getattr(recs[i], f) for f in REC_FIELDS) for i in range(m)]
    return {"records": out, "n_records": n.value, "counts": list(counts), "first_key": list(first),
            "site_stats": None}


def exec_kernel(text: str, launch, seed: int, *, input_mode=0, input_range=0, bits=32, checks=EQUIV | RACE | OOB,
                wmax=32, cap=1 << 22):
    """Run one kernel on one launch and seed; returns (init, final, counts) where
    init/final are lists of numpy arrays in global-id order (sorted array names)."""
    L = lib()
    lo = _launch(launch)
    init = (ctypes.c_uint32 * cap)()
    fin = (ctypes.c_uint32 * cap)()
    sizes = (ctypes.c_uint32 * 64)()
    na = ctypes.c_uint32(0)
    counts = (ctypes.c_int64 * 16)()
    rc = L.or_exec(text.encode(), ctypes.byref(lo), seed, input_mode, input_range, bits, checks, wmax, init, fin, cap,
                   sizes, 64, ctypes.byref(na), counts)
    if rc != 0:
        raise OracleError(rc, L.or_last_error().decode())
    a_init, a_fin, off = [], [], 0
    ai = np.ctypeslib.as_array(init)
    af = np.ctypeslib.as_array(fin)
    for g in range(na.value):
        n = sizes[g]
        a_init.append(ai[off:off + n].copy())
        a_fin.append(af[off:off + n].copy())
        off += n
    return a_init, a_fin, list(counts)


LOCK_FIELDS = ("launch", "seed_idx", "block", "round", "array", "addr", "val_src", "val_tgt", "written_src",
               "written_tgt")


def lockstep(src: str, tgt: str, launch_src, launch_tgt=None, *, lock_rounds=32, n_seeds=1, seed_base=0,
             input_mode=0, input_range=0, bits=32, cap=1 << 16):
    """Lock-step comparison of a pair (X25): per instance, the first (block, round,
    array, addr) at which the kernels' shared contents differ; rows of LOCK_FIELDS."""
    L = lib()
    ls = _launch_array(launch_src)
    lt = _launch_array(launch_tgt) if launch_tgt is not None else None
    sp = OrSpace()
    sp.launch_src = ctypes.cast(ls, ctypes.POINTER(OrLaunch))
    sp.launch_tgt = ctypes.cast(lt, ctypes.POINTER(OrLaunch)) if lt is not None else None
    sp.n_launch = len(launch_src)
    sp.seed_base, sp.n_seeds, sp.rank, sp.world = seed_base, n_seeds, 0, 1
    sp.input_mode, sp.input_range, sp.bits = input_mode, input_range, bits
    sp.checks, sp.wmax, sp.mode = EQUIV | RACE | OOB, 32, MODE_EQUIV
    rows = (ctypes.c_uint32 * (cap * 10))()
    n = ctypes.c_uint64(0)
    rc = L.or_lockstep(src.encode(), tgt.encode(), ctypes.byref(sp), lock_rounds, rows, cap, ctypes.byref(n))
    if rc != 0:
        raise OracleError(rc, L.or_last_error().decode())
    a = np.ctypeslib.as_array(rows)[: min(n.value, cap) * 10].reshape(-1, 10)
    return [tuple(int(x) for x in r) for r in a]


DF_FIELDS = ("block", "round", "gtid", "site", "array", "addr", "src_kind", "w_block", "w_round", "w_gtid")


def dataflow(text: str, launch, seed: int, *, bits=32, cap=1 << 20):
    """Data-flow relation (H5), cross-checked in VC-literal mode: rows of DF_FIELDS."""
    L = lib()
    lo = _launch(launch)
    rows = (ctypes.c_uint32 * (cap * 10))()
    n = ctypes.c_uint64(0)
    rc = L.or_dataflow(text.encode(), ctypes.byref(lo), seed, bits, rows, cap, ctypes.byref(n))
    if rc != 0:
        raise OracleError(rc, L.or_last_error().decode())
    a = np.ctypeslib.as_array(rows)[: min(n.value, cap) * 10].reshape(-1, 10)
    return [tuple(int(x) for x in r) for r in a]


def sm64(x: int) -> int:
    return lib().or_sm64(x)


def rand32(seed: int, tag: int, idx: int) -> int:
    return lib().or_rand32(seed, tag, idx)


def _check_shard(args):
    src, tgt, launch_src, launch_tgt, kw, rank, world = args
    return check(src, tgt, launch_src, launch_tgt, rank=rank, world=world, **kw)


def check_parallel(src: str, tgt, launch_src, launch_tgt=None, *, processes=0, **kw):
    """check() over host cores: one process per seed shard (the oracle's own rank/world
    sharding, seed j -> shard j mod world), results merged as H9 merges ranks - counts
    summed, first keys MIN, records (one per slot, so unique keys) in key order.  Test
    infrastructure, like check()."""
    import multiprocessing as mp
    n_seeds = kw.get("n_seeds", 1)
    world = max(1, min(processes or len(os.sched_getaffinity(0)), n_seeds))
    if kw.get("world", 1) != 1 or kw.get("rank", 0) != 0:
        raise ValueError("check_parallel shards by itself")
    kw = {k: v for k, v in kw.items() if k not in ("rank", "world")}
    build()
    if world == 1:
        return check(src, tgt, launch_src, launch_tgt, **kw)
    launch_src = [tuple(map(tuple, (l.gdim, l.bdim, l.scalars))) if hasattr(l, "gdim") else l for l in launch_src]
    if launch_tgt is not None:
        launch_tgt = [tuple(map(tuple, (l.gdim, l.bdim, l.scalars))) if hasattr(l, "gdim") else l
                      for l in launch_tgt]
    with mp.get_context("fork").Pool(world) as pool:
        parts = pool.map(_check_shard, [(src, tgt, launch_src, launch_tgt, kw, r, world) for r in range(world)])
    recs = sorted((r for p in parts for r in p["records"]), key=lambda r: r[0])
    counts = [sum(p["counts"][i] for p in parts) for i in range(16)]
    first = [min(p["first_key"][i] for p in parts) for i in range(11)]
    stats = None
    if parts[0]["site_stats"] is not None:
        stats = parts[0]["site_stats"].copy()
        for p in parts[1:]:
            s = p["site_stats"]
            stats[..., 0] = np.maximum(stats[..., 0], s[..., 0])
            stats[..., 3] = np.maximum(stats[..., 3], s[..., 3])
            for c in (1, 2, 4, 5, 6, 7):
                stats[..., c] += s[..., c]
    return {"records": recs, "n_records": sum(p["n_records"] for p in parts), "counts": counts,
            "first_key": first, "site_stats": stats}


def _check_n_shard(args):
    texts, launches, kw, rank, world = args
    return check_n(texts, launches, rank=rank, world=world, **kw)


def check_n_parallel(texts, launches, *, processes=0, **kw):
    """check_n() over host cores by seed shard, merged like check_parallel()."""
    import multiprocessing as mp
    n_seeds = kw.get("n_seeds", 1)
    world = max(1, min(processes or len(os.sched_getaffinity(0)), n_seeds))
    build()
    if world == 1:
        return check_n(texts, launches, **kw)
    launches = [[tuple(map(tuple, (l.gdim, l.bdim, l.scalars))) if hasattr(l, "gdim") else l for l in ls]
                for ls in launches]
    with mp.get_context("fork").Pool(world) as pool:
        parts = pool.map(_check_n_shard, [(texts, launches, kw, r, world) for r in range(world)])
    recs = sorted((r for p in parts for r in p["records"]), key=lambda r: r[0])
    return {"records": recs, "n_records": sum(p["n_records"] for p in parts),
            "counts": [sum(p["counts"][i] for p in parts) for i in range(16)],
            "first_key": [min(p["first_key"][i] for p in parts) for i in range(11)], "site_stats": None}
