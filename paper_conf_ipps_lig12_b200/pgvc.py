"""ctypes binding of libpgvc.so (include/pgvc.h) — argument marshalling only.

Every step of the checked path runs in the library's CUDA kernels; this module
only converts Python launch lists and torch tensors into the C structs.  It
loads the in-tree libpgvc.so and raises if it is missing: there is no CPU
fallback (use `python -m paper_conf_ipps_lig12_b200.build` to compile it).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass
from typing import List, Optional, Sequence

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libpgvc.so")

PG_OK, PG_E_ARG, PG_E_PARSE, PG_E_TYPE, PG_E_LIMIT, PG_E_CUDA, PG_E_OOM, PG_E_STATE = 0, -1, -2, -3, -4, -5, -6, -7
IN_RAND32, IN_BITS01, IN_RANGE = 0, 1, 2
CHK_EQUIV, CHK_RACE, CHK_OOB, CHK_BANK, CHK_COALESCE, CHK_DATAFLOW, CHK_LOCKSTEP, CHK_OPCOUNT = 1, 2, 4, 8, 16, 32, 64, 128
CHK_VCLITERAL = 256
LOCK_ROUNDS = 32
BANKS_32, BANKS_16_HALFWARP = 0, 1
KINDS = ["BARRIER_DIV", "OOB", "RACE_WW", "RACE_RW", "RACE_XB", "MISMATCH", "BANK", "UNCOALESCED", "UNINIT", "LIMIT"]
N_KINDS = 10
FAILING = {0, 1, 2, 3, 4, 5, 9}


class PgLaunch(ctypes.Structure):
    _fields_ = [("gdim", ctypes.c_uint32 * 3), ("bdim", ctypes.c_uint32 * 3), ("scalar", ctypes.c_int32 * 8),
                ("n_scalar", ctypes.c_uint32)]


class PgSpace(ctypes.Structure):
    _fields_ = [("launch_src", ctypes.POINTER(PgLaunch)), ("launch_tgt", ctypes.POINTER(PgLaunch)),
                ("n_launch", ctypes.c_uint32), ("seed_base", ctypes.c_uint64), ("n_seeds", ctypes.c_uint32),
                ("input_mode", ctypes.c_uint32), ("input_range", ctypes.c_uint32), ("bits", ctypes.c_uint32),
                ("checks", ctypes.c_uint32), ("bank_model", ctypes.c_uint32), ("max_cex", ctypes.c_uint32),
                ("rank", ctypes.c_int32), ("world", ctypes.c_int32), ("cuda_stream", ctypes.c_void_p),
                ("d_first_key", ctypes.c_void_p), ("d_counts", ctypes.c_void_p),
                ("key_launch0", ctypes.c_uint32), ("key_seed0", ctypes.c_uint32)]


LOCK_FIELDS = ("launch", "seed_idx", "block", "round", "array", "addr", "val_src", "val_tgt", "written_src",
               "written_tgt")
DF_FIELDS = ("launch", "seed_idx", "block", "round", "gtid", "site", "array", "addr", "src", "w_block",
             "w_round", "w_gtid")
REC_FIELDS = ("key", "count", "kind", "launch", "seed_idx", "kernel", "round", "site", "array", "addr",
              "tid_a", "tid_b", "val_a", "val_b")


class PgCex(ctypes.Structure):
    _fields_ = [("key", ctypes.c_uint64), ("count", ctypes.c_uint64)] + [
        (n, ctypes.c_uint32) for n in REC_FIELDS[2:]]


def _rec_dtype():
    import numpy as np
    return np.dtype([("key", "<u8"), ("count", "<u8")] + [(n, "<u4") for n in REC_FIELDS[2:]])


REC_DTYPE = _rec_dtype()


class PgSummary(ctypes.Structure):
    _fields_ = [("instances", ctypes.c_uint64), ("n_fail", ctypes.c_uint64), ("n_records", ctypes.c_uint64),
                ("first_key", ctypes.c_int64), ("first_launch", ctypes.c_uint32),
                ("first_seed_idx", ctypes.c_uint32), ("per_kind", ctypes.c_uint64 * N_KINDS),
                ("first_key_kind", ctypes.c_int64 * N_KINDS), ("ir_ops", ctypes.c_uint64)]


class PgError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__("pgvc error %d: %s" % (code, msg))
        self.code = code


_lib = None
EXPORTS = ["pg_load_ir", "pg_check_equiv", "pg_check_equiv_n", "pg_check_equiv_seq", "pg_check_races", "pg_check_banks", "pg_check_property", "pg_collect_cex",
           "pg_collect_site_stats", "pg_collect_dataflow", "pg_collect_lockstep", "pg_collect_vcliteral", "pg_ir_info",
           "pg_ir_seed_oblivious", "pg_ir_block_private", "pg_ir_thread_private",
           "pg_ir_source", "pg_ir_compile", "pg_run_timing", "pg_run_intervals", "pg_merge_counters",
           "pg_measure_int32_peak",
           "pg_last_error", "pg_ir_free", "pg_run_free", "pg_version"]


def lib():
    """Load the in-tree libpgvc.so (raises if it has not been built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError("libpgvc.so not built (run __graft_entry__.build() or python -m "
                          "paper_conf_ipps_lig12_b200.build); there is no CPU fallback")
    L = ctypes.CDLL(LIB_PATH)
    vp = ctypes.c_void_p
    L.pg_load_ir.argtypes = [ctypes.c_char_p, ctypes.c_size_t, ctypes.POINTER(vp)]
    L.pg_check_equiv.argtypes = [vp, vp, ctypes.POINTER(PgSpace), ctypes.POINTER(vp)]
    L.pg_check_races.argtypes = [vp, ctypes.POINTER(PgSpace), ctypes.POINTER(vp)]
    L.pg_check_equiv_n.argtypes = [ctypes.POINTER(vp), ctypes.c_uint32, ctypes.POINTER(ctypes.POINTER(PgLaunch)),
                                   ctypes.POINTER(PgSpace), ctypes.POINTER(vp)]
    L.pg_check_equiv_seq.argtypes = [ctypes.POINTER(vp), ctypes.c_uint32, ctypes.c_uint32,
                                     ctypes.POINTER(ctypes.POINTER(PgLaunch)), ctypes.POINTER(PgSpace),
                                     ctypes.POINTER(vp)]
    L.pg_check_banks.argtypes = [vp, ctypes.POINTER(PgSpace), ctypes.POINTER(vp)]
    L.pg_check_property.argtypes = [vp, vp, ctypes.POINTER(PgSpace), ctypes.POINTER(vp)]
    L.pg_collect_cex.argtypes = [vp, ctypes.POINTER(PgCex), ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t),
                                 ctypes.POINTER(PgSummary)]
    L.pg_collect_site_stats.argtypes = [vp, ctypes.POINTER(ctypes.c_uint64), ctypes.c_uint32]
    L.pg_collect_lockstep.argtypes = [vp, ctypes.POINTER(ctypes.c_uint32), ctypes.c_size_t,
                                      ctypes.POINTER(ctypes.c_size_t)]
    L.pg_collect_dataflow.argtypes = [vp, ctypes.POINTER(ctypes.c_uint32), ctypes.c_size_t,
                                      ctypes.POINTER(ctypes.c_size_t)]
    L.pg_collect_vcliteral.argtypes = [vp, ctypes.POINTER(ctypes.c_uint64)]
    L.pg_ir_info.argtypes = [vp, ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32),
                             ctypes.POINTER(ctypes.c_uint32)]
    L.pg_ir_seed_oblivious.argtypes = [vp, ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32)]
    L.pg_ir_block_private.argtypes = [vp, ctypes.POINTER(ctypes.c_uint32)]
    L.pg_ir_thread_private.argtypes = [vp, ctypes.POINTER(ctypes.c_uint64)]
    L.pg_ir_source.argtypes = [vp, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_char_p,
                               ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t)]
    L.pg_ir_compile.argtypes = [vp, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32]
    L.pg_run_timing.argtypes = [vp, ctypes.POINTER(ctypes.c_float), ctypes.POINTER(ctypes.c_float),
                                ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint64)]
    L.pg_run_intervals.argtypes = [vp, vp, ctypes.POINTER(ctypes.c_float), ctypes.c_size_t,
                                   ctypes.POINTER(ctypes.c_size_t)]
    L.pg_measure_int32_peak.argtypes = [vp, ctypes.POINTER(ctypes.c_double)]
    L.pg_merge_counters.argtypes = [vp, vp, ctypes.c_uint32, vp, vp, vp]
    L.pg_last_error.restype = ctypes.c_char_p
    L.pg_version.restype = ctypes.c_char_p
    L.pg_ir_free.argtypes = [vp]
    L.pg_run_free.argtypes = [vp]
    for f in ("pg_load_ir", "pg_check_equiv", "pg_check_equiv_n", "pg_check_equiv_seq", "pg_check_races", "pg_check_banks", "pg_check_property", "pg_collect_cex",
              "pg_collect_site_stats", "pg_collect_dataflow", "pg_collect_lockstep", "pg_collect_vcliteral",
              "pg_ir_info",
              "pg_ir_seed_oblivious", "pg_ir_block_private", "pg_ir_thread_private", "pg_ir_source", "pg_ir_compile", "pg_run_timing", "pg_run_intervals",
              "pg_merge_counters", "pg_measure_int32_peak"):
        getattr(L, f).restype = ctypes.c_int
    _lib = L
    return L


def _ck(rc: int):
    if rc != PG_OK:
        raise PgError(rc, lib().pg_last_error().decode())


class Ir:
    """A loaded kernel (pg_load_ir)."""

    def __init__(self, text: str):
        self.text = text
        self._h = ctypes.c_void_p()
        b = text.encode()
        _ck(lib().pg_load_ir(b, len(b), ctypes.byref(self._h)))

    @property
    def handle(self):
        return self._h

    def info(self):
        s, g, c = ctypes.c_uint32(), ctypes.c_uint32(), ctypes.c_uint32()
        _ck(lib().pg_ir_info(self._h, ctypes.byref(s), ctypes.byref(g), ctypes.byref(c)))
        return {"sites": s.value, "globals": g.value, "scalars": c.value}

    def seed_oblivious(self):
        """(oblivious, n_tainted): pg_ir_seed_oblivious."""
        o, n = ctypes.c_uint32(), ctypes.c_uint32()
        _ck(lib().pg_ir_seed_oblivious(self._h, ctypes.byref(o), ctypes.byref(n)))
        return bool(o.value), n.value

    def block_private(self) -> bool:
        """pg_ir_block_private: every written global array is write-only at index bid.x."""
        b = ctypes.c_uint32()
        _ck(lib().pg_ir_block_private(self._h, ctypes.byref(b)))
        return bool(b.value)

    def thread_private(self) -> int:
        """pg_ir_thread_private: bit a = array a's stores are all at index tid.x."""
        m = ctypes.c_uint64()
        _ck(lib().pg_ir_thread_private(self._h, ctypes.byref(m)))
        return m.value

    def source(self, bits=32, checks=CHK_RACE | CHK_OOB, bank_model=0) -> str:
        n = ctypes.c_size_t()
        _ck(lib().pg_ir_source(self._h, bits, checks, bank_model, None, 0, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value + 1)
        _ck(lib().pg_ir_source(self._h, bits, checks, bank_model, buf, n.value + 1, ctypes.byref(n)))
        return buf.value.decode()

    def compile(self, bits=32, checks=CHK_RACE | CHK_OOB, bank_model=0):
        _ck(lib().pg_ir_compile(self._h, bits, checks, bank_model))

    def __del__(self):
        if getattr(self, "_h", None) and self._h.value and _lib is not None:
            _lib.pg_ir_free(self._h)
            self._h = ctypes.c_void_p()


def load_ir(text: str) -> Ir:
    return Ir(text)


def _launch(l) -> PgLaunch:
    gdim, bdim, sc = (l.gdim, l.bdim, l.scalars) if hasattr(l, "gdim") else l
    o = PgLaunch()
    for i in range(3):
        o.gdim[i] = gdim[i]
        o.bdim[i] = bdim[i]
    for i, v in enumerate(sc):
        o.scalar[i] = v
    o.n_scalar = len(sc)
    return o


def _counter_ptr(t, n: int, what: str):
    """Device pointer of a caller-owned counter tensor (pg_space.d_first_key / d_counts):
    the library writes n int64 values through it, so it must be a contiguous int64 CUDA
    tensor of >= n elements on the current device."""
    if t is None:
        return None
    import torch
    ok = (isinstance(t, torch.Tensor) and t.device.type == "cuda" and t.dtype == torch.int64
          and t.is_contiguous() and t.numel() >= n and t.device.index == torch.cuda.current_device())
    if not ok:
        raise PgError(PG_E_ARG, "%s must be a contiguous int64 CUDA tensor of >= %d elements on the current "
                                "device" % (what, n))
    return t.data_ptr()


@dataclass
class Space:
    """Python side of pg_space.  Launches are Launch objects or (gdim, bdim, scalars)."""
    launch_src: Sequence
    launch_tgt: Optional[Sequence] = None
    n_seeds: int = 1
    seed_base: int = 0
    input_mode: int = IN_RAND32
    input_range: int = 0
    bits: int = 32
    checks: int = CHK_EQUIV | CHK_RACE | CHK_OOB
    bank_model: int = BANKS_32
    max_cex: int = 1 << 20
    rank: int = 0
    world: int = 1
    stream: int = 0                 # cudaStream_t as an integer (torch.cuda.Stream.cuda_stream)
    first_key: object = None        # torch int64[11] on the device (optional)
    counts: object = None           # torch int64[16] on the device (optional)
    key_launch0: int = 0            # launch / seed index offsets of the keys (a sub-space of a larger space)
    key_seed0: int = 0

    def marshal(self):
        # (the launch arrays are built once per Space object: a Space re-used for every step
        # of a loop marshals its launch lists once)
        key = (id(self.launch_src), len(self.launch_src), id(self.launch_tgt))
        cached = self.__dict__.get("_launch_arrays")
        if cached is not None and cached[0] == key:
            ls, lt = cached[1], cached[2]
        else:
            ls = (PgLaunch * max(1, len(self.launch_src)))(*[_launch(l) for l in self.launch_src])
            lt = None
            if self.launch_tgt is not None:
                lt = (PgLaunch * max(1, len(self.launch_tgt)))(*[_launch(l) for l in self.launch_tgt])
            self.__dict__["_launch_arrays"] = (key, ls, lt)
        sp = PgSpace()
        sp.launch_src = ctypes.cast(ls, ctypes.POINTER(PgLaunch))
        sp.launch_tgt = ctypes.cast(lt, ctypes.POINTER(PgLaunch)) if lt is not None else None
        sp.n_launch = len(self.launch_src)
        sp.seed_base = self.seed_base
        sp.n_seeds = self.n_seeds
        sp.input_mode, sp.input_range, sp.bits = self.input_mode, self.input_range, self.bits
        sp.checks, sp.bank_model, sp.max_cex = self.checks, self.bank_model, self.max_cex
        sp.rank, sp.world = self.rank, self.world
        sp.cuda_stream = self.stream or None
        sp.d_first_key = _counter_ptr(self.first_key, 11, "first_key")
        sp.d_counts = _counter_ptr(self.counts, 16, "counts")
        sp.key_launch0, sp.key_seed0 = self.key_launch0, self.key_seed0
        return sp, (ls, lt)


class Run:
    """Result set of one check (pg_run).  collect() synchronises its stream."""

    def __init__(self, h, space: Space, keep):
        self._h = h
        self.space = space
        self._keep = keep

    def collect(self, cap: int = 1 << 20, tuples: bool = True):
        """Synchronise, copy up to `cap` records.  Returns (records, summary): records as a
        list of tuples in REC_FIELDS order (tuples=True) or a numpy structured array."""
        import numpy as np
        n = ctypes.c_size_t()
        summ = PgSummary()
        buf = np.empty(max(1, cap), dtype=REC_DTYPE)
        _ck(lib().pg_collect_cex(self._h, buf.ctypes.data_as(ctypes.POINTER(PgCex)), cap, ctypes.byref(n),
                                 ctypes.byref(summ)))
        arr = buf[:min(n.value, cap, self.space.max_cex or (1 << 20))]   # the run keeps max_cex
        recs = arr.tolist() if tuples else arr
        s = {"instances": summ.instances, "n_fail": summ.n_fail, "n_records": summ.n_records, "n_local": n.value,
             "first_key": summ.first_key, "first_launch": summ.first_launch,
             "first_seed_idx": summ.first_seed_idx, "per_kind": list(summ.per_kind),
             "first_key_kind": list(summ.first_key_kind), "ir_ops": summ.ir_ops}
        return recs, s

    def site_stats(self, max_sites: int):
        import numpy as np
        nl = len(self.space.launch_src)
        out = np.zeros((nl, 2, max_sites, 8), dtype=np.uint64)
        _ck(lib().pg_collect_site_stats(self._h, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), max_sites))
        return out

    def dataflow(self):
        """Data-flow rows of a run checked with CHK_DATAFLOW: uint32 array (n, 12) in
        DF_FIELDS order, sorted lexicographically."""
        import numpy as np
        n = ctypes.c_size_t()
        _ck(lib().pg_collect_dataflow(self._h, None, 0, ctypes.byref(n)))
        out = np.zeros((max(1, n.value), 12), dtype=np.uint32)
        _ck(lib().pg_collect_dataflow(self._h, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)), n.value,
                                      ctypes.byref(n)))
        out = out[:min(n.value, 1 << 20)]
        return out[np.lexsort(out.T[::-1])] if len(out) else out

    def vcliteral(self):
        """(reads checked literally, disagreements with the owner-stamp writer, history
        overflows) of a CHK_VCLITERAL run (pg_collect_vcliteral)."""
        out = (ctypes.c_uint64 * 3)()
        _ck(lib().pg_collect_vcliteral(self._h, out))
        return {"checked": out[0], "disagree": out[1], "overflow": out[2]}

    def lockstep(self):
        """First shared-state divergence per instance of a PG_CHK_LOCKSTEP equivalence run:
        list of tuples in LOCK_FIELDS order, (launch, seed) order."""
        import numpy as np
        n = ctypes.c_size_t()
        _ck(lib().pg_collect_lockstep(self._h, None, 0, ctypes.byref(n)))
        out = np.zeros((max(1, n.value), 10), dtype=np.uint32)
        _ck(lib().pg_collect_lockstep(self._h, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)), n.value,
                                      ctypes.byref(n)))
        return [tuple(int(x) for x in r) for r in out[:n.value]]

    def timing(self):
        a, b, n, h = ctypes.c_float(), ctypes.c_float(), ctypes.c_uint32(), ctypes.c_uint64()
        _ck(lib().pg_run_timing(self._h, ctypes.byref(a), ctypes.byref(b), ctypes.byref(n), ctypes.byref(h)))
        return {"ms_eval": a.value, "ms_total": b.value, "launches": n.value, "h2d_bytes": h.value}

    def intervals(self, ref_event=None):
        """[(start_ms, end_ms)] of every evaluation-kernel launch of the run, relative to
        ref_event (a torch.cuda.Event recorded before the check) or to the run's first
        enqueued operation (pg_run_intervals)."""
        ref = ctypes.c_void_p(ref_event.cuda_event) if ref_event is not None else None
        n = ctypes.c_size_t()
        _ck(lib().pg_run_intervals(self._h, ref, None, 0, ctypes.byref(n)))
        buf = (ctypes.c_float * max(2, 2 * n.value))()
        _ck(lib().pg_run_intervals(self._h, ref, buf, n.value, ctypes.byref(n)))
        return [(buf[2 * i], buf[2 * i + 1]) for i in range(n.value)]

    def __del__(self):
        if getattr(self, "_h", None) and self._h.value and _lib is not None:
            _lib.pg_run_free(self._h)
            self._h = ctypes.c_void_p()


def _run(fn, irs, space: Space) -> Run:
    sp, keep = space.marshal()
    h = ctypes.c_void_p()
    _ck(fn(*[i.handle for i in irs], ctypes.byref(sp), ctypes.byref(h)))
    return Run(h, space, (keep, irs))


def pg_check_equiv(src: Ir, tgt: Ir, space: Space) -> Run:
    return _run(lib().pg_check_equiv, [src, tgt], space)


def _launch_ptrs(space: Space, launches, tag: str):
    n = len(launches[0])
    if any(len(l) != n for l in launches):
        raise PgError(PG_E_ARG, "launch lists of different lengths")
    key = (id(launches), len(launches), n)
    cached = space.__dict__.get(tag)   # (marshalled once per Space object, as marshal() does)
    if cached is not None and cached[0] == key:
        return n, cached[1], cached[2]
    arrs = [(PgLaunch * max(1, n))(*[_launch(l) for l in ls]) for ls in launches]
    ptrs = (ctypes.POINTER(PgLaunch) * len(arrs))(*[ctypes.cast(a, ctypes.POINTER(PgLaunch)) for a in arrs])
    space.__dict__[tag] = (key, arrs, ptrs)
    return n, arrs, ptrs


def pg_check_equiv_seq(src: Sequence[Ir], tgt: Sequence[Ir], src_launches: Sequence[Sequence],
                       tgt_launches: Sequence[Sequence], space: Space) -> Run:
    """Kernel sequences (pg_check_equiv_seq): the source kernels run in order on one set of
    global buffers, so do the target kernels; final buffers compared.  *_launches[i] is
    phase i's launch list."""
    kernels = list(src) + list(tgt)
    if len(src) < 1 or len(tgt) < 1 or len(kernels) > 8:
        raise PgError(PG_E_ARG, "1 to 7 kernels per side, 8 in all")
    launches = list(src_launches) + list(tgt_launches)
    if len(launches) != len(kernels):
        raise PgError(PG_E_ARG, "one launch list per kernel")
    sp, keep = space.marshal()
    n, arrs, ptrs = _launch_ptrs(space, launches, "_seq_arrays")
    sp.launch_src = ptrs[0]
    sp.launch_tgt = None
    sp.n_launch = n
    hs = (ctypes.c_void_p * len(kernels))(*[k.handle.value for k in kernels])
    h = ctypes.c_void_p()
    _ck(lib().pg_check_equiv_seq(hs, len(kernels), len(src), ptrs, ctypes.byref(sp), ctypes.byref(h)))
    return Run(h, space, (keep, arrs, ptrs, kernels))


def pg_check_equiv_n(kernels: Sequence[Ir], launches: Sequence[Sequence], space: Space) -> Run:
    """Every kernel once per (launch, seed), every pair compared (pg_check_equiv_n).
    launches[k]: kernel k's launch list (same length for all); space.launch_src is ignored
    except as the list length / fallback (pass launches[0])."""
    if not 2 <= len(kernels) <= 8 or len(launches) != len(kernels):
        raise PgError(PG_E_ARG, "2 to 8 kernels, one launch list each")
    n = len(launches[0])
    if any(len(l) != n for l in launches):
        raise PgError(PG_E_ARG, "launch lists of different lengths")
    sp, keep = space.marshal()
    key = (id(launches), len(launches), n)
    cached = space.__dict__.get("_n_arrays")   # (marshalled once per Space object, as marshal() does)
    if cached is not None and cached[0] == key:
        arrs, ptrs = cached[1], cached[2]
    else:
        arrs = [(PgLaunch * max(1, n))(*[_launch(l) for l in ls]) for ls in launches]
        ptrs = (ctypes.POINTER(PgLaunch) * len(arrs))(*[ctypes.cast(a, ctypes.POINTER(PgLaunch)) for a in arrs])
        space.__dict__["_n_arrays"] = (key, arrs, ptrs)
    sp.launch_src = ptrs[0]
    sp.launch_tgt = None
    sp.n_launch = n
    hs = (ctypes.c_void_p * len(kernels))(*[k.handle.value for k in kernels])
    h = ctypes.c_void_p()
    _ck(lib().pg_check_equiv_n(hs, len(kernels), ptrs, ctypes.byref(sp), ctypes.byref(h)))
    return Run(h, space, (keep, arrs, ptrs, kernels))


def pg_check_races(k: Ir, space: Space) -> Run:
    return _run(lib().pg_check_races, [k], space)


def pg_check_banks(k: Ir, space: Space) -> Run:
    return _run(lib().pg_check_banks, [k], space)


def pg_check_property(k: Ir, post: Ir, space: Space) -> Run:
    """k against the post-condition kernel `post` (one thread per launch; see pgvc.h)."""
    if space.launch_tgt is not None:
        raise ValueError("property mode derives the post-condition launches; launch_tgt must be None")
    return _run(lib().pg_check_property, [k, post], space)


check_equiv, check_races, check_banks, check_property = pg_check_equiv, pg_check_races, pg_check_banks, pg_check_property
check_equiv_n, check_equiv_seq = pg_check_equiv_n, pg_check_equiv_seq


def merge_counters(first_keys, counts, out_first_key, out_counts, stream: int = 0):
    """pg_merge_counters: MIN over the rows of first_keys (n x 11), SUM over the rows of counts
    (n x 16), into out_first_key (11) / out_counts (16); int64 CUDA tensors."""
    n = first_keys.shape[0]
    if counts.shape[0] != n or first_keys.shape[1:] != (11,) or counts.shape[1:] != (16,):
        raise PgError(PG_E_ARG, "first_keys must be (n, 11) and counts (n, 16)")
    _ck(lib().pg_merge_counters(ctypes.c_void_p(_counter_ptr(first_keys, 11 * n, "first_keys")),
                                ctypes.c_void_p(_counter_ptr(counts, 16 * n, "counts")), n,
                                ctypes.c_void_p(_counter_ptr(out_first_key, 11, "out_first_key")),
                                ctypes.c_void_p(_counter_ptr(out_counts, 16, "out_counts")),
                                ctypes.c_void_p(stream or None)))


def measure_int32_peak(stream: int = 0):
    """Integer ops/s of the current device (pg_measure_int32_peak): alu pipe (LOP3),
    fma pipe (IMAD), both pipes alternating."""
    out = (ctypes.c_double * 3)()
    _ck(lib().pg_measure_int32_peak(ctypes.c_void_p(stream or None), out))
    return {"alu": out[0], "fma": out[1], "mixed": out[2]}


def version() -> str:
    return lib().pg_version().decode()
