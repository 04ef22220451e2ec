"""Seeded, synthetic workload definitions (the bounded parameter spaces C1-C5).

INPUT GENERATION ONLY.  This module holds none of the method's arithmetic: it
only lists launches (gdim, bdim, scalar parameters) in witness order and names
subject kernel files.  It is the one module both the CUDA path and the oracle
tests draw their inputs from (the per-cell input VALUES are generated
independently on each side from the counter-based PRF of DESIGN.md X8).

Each config follows SURVEY.md §8(d) and BASELINE.json `configs`:
  C1  naive vs shared-memory transpose, bdim in [1,4]^2, up to 16x16 threads
      (the Table II transpose rows L909-L911)
  C2  reduce0..reduce6 pairwise equivalence (L825-L837 + SDK reduction)
  C3  Blelloch exclusive scan vs bank-conflict-free padded scan
  C4  bitonic sort global vs shared
  C5  32x32 tiled transpose and matrix multiply
"""
from __future__ import annotations

import os
from dataclasses import dataclass, field
from typing import List, Sequence, Tuple

SUBJECT_DIR = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "subjects")


@dataclass(frozen=True)
class Launch:
    """One value of the parameter n: grid and block shape plus scalar params."""
    gdim: Tuple[int, int, int]
    bdim: Tuple[int, int, int]
    scalars: Tuple[int, ...] = ()

    @property
    def threads_per_block(self) -> int:
        return self.bdim[0] * self.bdim[1] * self.bdim[2]

    @property
    def blocks(self) -> int:
        return self.gdim[0] * self.gdim[1] * self.gdim[2]

    @property
    def threads(self) -> int:
        return self.threads_per_block * self.blocks


def subject(name: str) -> str:
    """Text of subjects/<name>.pgk."""
    with open(os.path.join(SUBJECT_DIR, name + ".pgk")) as f:
        return f.read()


@dataclass
class Workload:
    name: str
    src: str                       # subject file stem of the source kernel
    tgt: str                       # subject file stem of the target kernel ("" for single-kernel checks)
    launch_src: List[Launch]
    launch_tgt: List[Launch]
    n_seeds: int = 64
    seed_base: int = 0
    input_mode: int = 0            # 0 RAND32, 1 BITS01, 2 RANGE
    input_range: int = 0
    checks: int = 1 | 2 | 4        # EQUIV | RACE | OOB
    note: str = ""
    extra: dict = field(default_factory=dict)


# ---------------------------------------------------------------- C1
def c1_launches(max_side: int = 16, max_b: int = 4, ragged: bool = False) -> List[Launch]:
    """C1: bdim (bx,by) in [1,max_b]^2, gx*bx <= 16, gy*by <= 16,
    width = gx*bx, height = gy*by (exact cover); ordered by
    (total threads, by, bx, gy, gx) = witness order (X16).
    ragged=True adds width-1 / height-1 variants (tests only)."""
    out = []
    for bx in range(1, max_b + 1):
        for by in range(1, max_b + 1):
            for gx in range(1, max_side // bx + 1):
                for gy in range(1, max_side // by + 1):
                    w, h = gx * bx, gy * by
                    sizes = [(w, h)]
                    if ragged:
                        sizes += [(w - 1, h), (w, h - 1)]
                    for (ww, hh) in sizes:
                        if ww < 1 or hh < 1:
                            continue
                        out.append((bx * by * gx * gy, by, bx, gy, gx, ww, hh))
    out.sort()
    return [Launch((gx, gy, 1), (bx, by, 1), (w, h)) for (_, by, bx, gy, gx, w, h) in out]


def c1(n_seeds: int = 64) -> Workload:
    ls = c1_launches()
    return Workload("C1", "naive_transpose", "optimized_transpose", ls, ls, n_seeds=n_seeds,
                    note="naive vs shared-mem transpose, 4x4 tiles, n up to 16x16 threads")


def pack_launches(ls: Sequence[Launch]):
    """Flatten launches to plain tuples (gdim, bdim, scalars) for the C bindings."""
    return [(tuple(l.gdim), tuple(l.bdim), tuple(l.scalars)) for l in ls]


# ---------------------------------------------------------------- C2
REDUCE_HALF = {"reduce3", "reduce4", "reduce5", "reduce6", "reduce4_warpsync"}


def reduce_launch(kernel: str, N: int, B: int) -> Launch:
    """Launch of one SDK reduction variant reducing B elements per block, N total:
    reduce0-2 use bdim = B, reduce3-6 bdim = B/2 (2 elements per thread); gdim = N/B
    for all, so g_odata[b] = sum(g_idata[bB:(b+1)B]) in every variant."""
    bd = B // 2 if kernel in REDUCE_HALF else B
    if kernel in ("reduce4", "reduce5", "reduce4_warpsync"):
        sc = (N, bd)
    elif kernel == "reduce6":
        sc = (N, bd, 1 if (N & (N - 1)) == 0 else 0)
    else:
        sc = (N,)
    return Launch((N // B, 1, 1), (bd, 1, 1), sc)


def c2_points(max_log_n: int = 16, max_log_b: int = 10, min_log_b: int = 0):
    """(N, B) with B = 2^0..2^10 and N = B..2^16 powers of two, ordered by (N, B)."""
    pts = []
    for lb in range(min_log_b, max_log_b + 1):
        for ln in range(lb, max_log_n + 1):
            pts.append((1 << ln, 1 << lb))
    pts.sort()
    return pts


C2_PAIRS = [("reduce0", "reduce1"), ("reduce0", "reduce2"), ("reduce0", "reduce3"), ("reduce0", "reduce4"),
            ("reduce0", "reduce5"), ("reduce0", "reduce6"), ("reduce2", "reduce2_obo")]


def c2_pair(src: str, tgt: str, n_seeds: int = 64, max_log_n: int = 16, max_log_b: int = 10) -> Workload:
    min_lb = 1 if (src in REDUCE_HALF or tgt in REDUCE_HALF) else 0
    pts = c2_points(max_log_n, max_log_b, min_lb)
    return Workload("C2:%s-%s" % (src, tgt), src, tgt, [reduce_launch(src, N, B) for N, B in pts],
                    [reduce_launch(tgt, N, B) for N, B in pts], n_seeds=n_seeds,
                    note="SDK reduction variants, blockDim up to 1024, n up to 2^16")


def c2(n_seeds: int = 64, max_log_n: int = 16, max_log_b: int = 10) -> List[Workload]:
    return [c2_pair(s, t, n_seeds, max_log_n, max_log_b) for s, t in C2_PAIRS]


C2_ALL = ["reduce0", "reduce1", "reduce2", "reduce3", "reduce4", "reduce5", "reduce6", "reduce2_obo"]


@dataclass
class NWorkload:
    """An N-kernel check (pg_check_equiv_n): kernels[k] with launch list launches[k]."""
    name: str
    kernels: List[str]
    launches: List[List[Launch]]
    n_seeds: int = 64
    checks: int = 7


def c2_all(n_seeds: int = 64, max_log_n: int = 16, max_log_b: int = 10) -> List[NWorkload]:
    """SURVEY.md §8(d)'s C2 design: reduce0..reduce6 and the injected off-by-one, each
    evaluated once per (N, B, seed), every pair compared (28 pairs).  B = 1 has no
    reduce3..6 launch (B/2 threads), so its points form a second check of the four
    B-thread kernels."""
    full = c2_points(max_log_n, max_log_b, 1)
    b1 = [(N, B) for N, B in c2_points(max_log_n, max_log_b, 0) if B == 1]
    four = ["reduce0", "reduce1", "reduce2", "reduce2_obo"]
    return [NWorkload("C2:all", list(C2_ALL), [[reduce_launch(k, N, B) for N, B in full] for k in C2_ALL], n_seeds),
            NWorkload("C2:B=1", four, [[reduce_launch(k, N, B) for N, B in b1] for k in four], n_seeds)]


# ---------------------------------------------------------------- C3
def scan_launch(kernel: str, n: int, B: int, lognb: int = 4) -> Launch:
    sc = (n, lognb) if kernel == "prescan_padded" else (n,)
    return Launch((n // (2 * B), 1, 1), (B, 1, 1), sc)


def c3_points(max_log_n: int = 14, max_log_b: int = 10):
    """(n, B): B = 2^0..2^10 threads, 2B elements per block, n = G*2B <= 2^14, order (n, B)."""
    pts = []
    for lb in range(0, max_log_b + 1):
        for ln in range(lb + 1, max_log_n + 1):
            pts.append((1 << ln, 1 << lb))
    pts.sort()
    return pts


def c3_pair(tgt: str = "prescan_padded", lognb: int = 4, n_seeds: int = 64, max_log_n: int = 14,
            max_log_b: int = 10) -> Workload:
    pts = c3_points(max_log_n, max_log_b)
    return Workload("C3:prescan-%s%s" % (tgt, "" if tgt != "prescan_padded" else str(lognb)), "prescan", tgt,
                    [scan_launch("prescan", n, B) for n, B in pts],
                    [scan_launch(tgt, n, B, lognb) for n, B in pts], n_seeds=n_seeds,
                    checks=1 | 2 | 4 | 8 | 16, note="Blelloch scan vs padded scan, n up to 2^14")


# ---------------------------------------------------------------- C4
def bitonic_launch(kernel: str, n: int) -> Launch:
    return Launch((1, 1, 1), (n if kernel == "bitonic_global" else n // 2, 1, 1), (n,))


def c4(mode: str = "rand", n_seeds: int = 64, max_log_n: int = 12) -> List[Workload]:
    """mode 'rand': RAND32 x n_seeds; 'range': RANGE(4) x n_seeds (ties);
    'bits': BITS01 exhaustive 2^n seeds, one workload per n <= 16 (0-1 principle)."""
    out = []
    if mode == "bits":
        for ln in range(1, min(max_log_n, 4) + 1):
            n = 1 << ln
            out.append(Workload("C4:bits%d" % n, "bitonic_global", "bitonic_shared",
                                [bitonic_launch("bitonic_global", n)], [bitonic_launch("bitonic_shared", n)],
                                n_seeds=1 << n, input_mode=1))
        return out
    ns = [1 << ln for ln in range(1, max_log_n + 1)]
    out.append(Workload("C4:" + mode, "bitonic_global", "bitonic_shared",
                        [bitonic_launch("bitonic_global", n) for n in ns],
                        [bitonic_launch("bitonic_shared", n) for n in ns], n_seeds=n_seeds,
                        input_mode=2 if mode == "range" else 0, input_range=4 if mode == "range" else 0))
    return out


# ---------------------------------------------------------------- C5
def c5_transpose(n_seeds: int = 10000, sizes=(32, 64, 128, 256, 512, 1024), tgt: str = "optimized_transpose",
                 tile: int = 32) -> Workload:
    ls = [Launch((N // tile, N // tile, 1), (tile, tile, 1), (N, N)) for N in sizes]
    return Workload("C5:transpose", "naive_transpose", tgt, ls, ls, n_seeds=n_seeds,
                    note="tiled 32x32 transpose, 2D grids up to 1024x1024 threads")


def c5_matmul(n_seeds: int = 10000, sizes=(32, 64, 128, 256, 512, 1024), K: int = 64,
              tgt: str = "matmul_tiled", tile: int = 32) -> Workload:
    ls = [Launch((N // tile, N // tile, 1), (tile, tile, 1), (K, N, N)) for N in sizes]
    return Workload("C5:matmul", "matmul_naive", tgt, ls, ls, n_seeds=n_seeds,
                    note="naive vs tiled matmul, K = %d" % K)


# ---------------------------------------------------------------- property mode (NEXT-1)
POST = {"reduce": "post_reduce", "scan": "post_scan", "transpose": "post_transpose"}


def property_launches(launches: Sequence[Launch], n_post_scalars: int) -> List[Launch]:
    """The post-condition launches pg_check_property derives (include/pgvc.h): one block of
    one thread whose scalars are the first m of (gdim.x, gdim.y, bdim.x, bdim.y, scalars)."""
    out = []
    for l in launches:
        v = (l.gdim[0], l.gdim[1], l.bdim[0], l.bdim[1]) + tuple(l.scalars)
        assert n_post_scalars <= len(v)
        out.append(Launch((1, 1, 1), (1, 1, 1), tuple(v[:n_post_scalars])))
    return out


# ---------------------------------------------------------------- configuration bugs (NEXT-3)
def scalar_prod_launch(vectorN: int, elementN: int, accn: int, bdim: int) -> Launch:
    """scalarProd with one vector per block (gdim.x = vectorN), ACCN partial sums."""
    return Launch((vectorN, 1, 1), (bdim, 1, 1), (vectorN, elementN, accn))


def accn_sweep(max_accn: int = 16, bdims=(1, 4, 8), vectorN: int = 2, elementN: int = 40) -> List[Launch]:
    """ACCN = 1..max_accn in order (the witness order), for each block size."""
    return [scalar_prod_launch(vectorN, elementN, a, b) for a in range(1, max_accn + 1) for b in bdims]


@dataclass
class SeqWorkload:
    """A sequence check (pg_check_equiv_seq): the source kernels run in order on one set of
    global buffers, so do the target kernels; launches[i] is phase i's launch list."""
    name: str
    src: List[str]
    tgt: List[str]
    src_launches: List[List[Launch]]
    tgt_launches: List[List[Launch]]
    n_seeds: int = 64
    checks: int = 7


def reduce_two_pass(n_seeds: int = 8, max_log_n: int = 14, max_log_b: int = 10, first: str = "reduce0",
                    second: str = "reduce0_pass2") -> SeqWorkload:
    """The SDK's multi-pass reduction as a kernel sequence (GKLEE multi-kernel programs,
    PAPER.md L62-L63): `first` reduces N inputs to M = N/B block sums (g_odata), `second`
    reduces those in one block of M threads into g_sum[0]; the target is the one-thread
    specification sum_serial.  Points (N, B) with M = N/B <= 1024, powers of two."""
    pts = [(N, B) for N, B in c2_points(max_log_n, max_log_b, 0) if N // B <= 1024]
    p1 = [reduce_launch(first, N, B) for N, B in pts]
    p2 = [Launch((1, 1, 1), (N // B, 1, 1), (N // B,)) for N, B in pts]
    ser = [Launch((1, 1, 1), (1, 1, 1), (N,)) for N, B in pts]
    return SeqWorkload("C2:two-pass", [first, second], ["sum_serial"], [p1, p2], [ser], n_seeds)
