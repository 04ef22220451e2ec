"""Oracle pins for matmul and the 32x32 tile bank/coalescing facts (SURVEY.md P6 and the
hand-derivable textbook values, ref [8])."""
import numpy as np
import pytest


def mm(A, B, n, k, m):
    return ((A.astype(object).reshape(n, k).dot(B.astype(object).reshape(k, m))) % (1 << 32)).astype(np.uint32)


@pytest.mark.parametrize("name", ["matmul_naive", "matmul_tiled"])
def test_closed_form_product(oracle, W, name):
    # C = A B mod 2^32 (triple loop); gid order: A, B, C
    for N, K, t in [(4, 4, 4), (8, 12, 4), (16, 8, 8)]:
        l = ((N // t, N // t, 1), (t, t, 1), (K, N, N))
        _, fin, counts = oracle.exec_kernel(W.subject(name), l, 5)
        assert (fin[2] == mm(fin[0], fin[1], N, K, N).reshape(-1)).all()
        assert sum(counts[1:11]) == 0


def test_dropped_trailing_barrier(oracle, W):
    # P6: without the trailing barrier the next tile's loads race with this tile's reads (RW),
    # first at wA = 2 tiles; outputs stay equal under X3 (reads precede the thread's own next writes)
    t, N = 4, 8
    for K, racy in ((4, False), (8, True), (12, True)):
        l = ((N // t, N // t, 1), (t, t, 1), (K, N, N))
        r = oracle.check(W.subject("matmul_tiled"), W.subject("matmul_tiled_nobarrier"), [l], [l], n_seeds=2)
        kinds = {x[2] for x in r["records"]}
        assert (3 in kinds) == racy and 5 not in kinds


def test_dropped_middle_barrier(oracle, W):
    # P6: without the barrier between tile load and use, a thread reads tile cells other threads
    # write in the same round: race and wrong C at any K >= TILE
    text = W.subject("matmul_tiled")
    i = text.index("sync;")
    broken = text[:i] + text[i + len("sync;"):]
    t, N, K = 4, 8, 4
    l = ((N // t, N // t, 1), (t, t, 1), (K, N, N))
    r = oracle.check(text, broken, [l], [l], n_seeds=1)
    kinds = {x[2] for x in r["records"]}
    assert 3 in kinds and 5 in kinds


def site_rows(oracle, text, launch):
    r = oracle.check(text, None, [launch], mode=2, checks=oracle.BANK | oracle.COALESCE, max_sites=16)
    return r["site_stats"][0, 0]


def test_tile_bank_conflicts_32x32(oracle, W):
    # unpadded [32][32] column read block[tid.x][tid.y]: 32 lanes, one bank -> degree 32;
    # padded [32][33]: bank (33 tx + ty) mod 32 all distinct -> degree 1 (L155's "+1")
    l = ((1, 1, 1), (32, 32, 1), (32, 32))
    un = site_rows(oracle, W.subject("optimized_transpose_unpadded"), l)
    pd = site_rows(oracle, W.subject("optimized_transpose"), l)
    # sites: 0 block store, 1 idata load, 2 sync, 3 odata store, 4 block load
    assert un[4][0] == 1 and un[4][3] == 32 and un[4][1] == 32 and un[4][2] == 32
    assert pd[4][3] == 1 and pd[4][2] == 0
    assert un[0][3] == 1 and pd[0][3] == 1


def test_transpose_coalescing_32x32(oracle, W):
    # naive write odata[y + height*x]: 32 lanes at stride height -> 32 sectors (ideal 4); its read and
    # both optimized global accesses are 32 consecutive words -> 4 sectors = ideal (L146-L150)
    l = ((1, 1, 1), (32, 32, 1), (32, 32))
    nv = site_rows(oracle, W.subject("naive_transpose"), l)
    op = site_rows(oracle, W.subject("optimized_transpose"), l)
    # naive sites: 0 odata store, 1 idata load
    assert nv[0][0] == 2 and nv[0][3] == 32 and nv[0][2] == 32 and nv[0][5] == 32 * 4
    assert nv[1][3] == 4 and nv[1][2] == 0
    assert op[1][3] == 4 and op[3][3] == 4 and op[1][2] == 0 and op[3][2] == 0


def test_c1_tiles_show_no_coalescing_difference(oracle, W):
    # at 4x4 tiles (C1, 16x16 matrix) a warp is one 16-thread block: both kernels' odata writes
    # touch 4 sectors against an ideal of 2 (SURVEY.md §8(c) last pin row)
    l = ((4, 4, 1), (4, 4, 1), (16, 16))
    nv = site_rows(oracle, W.subject("naive_transpose"), l)
    op = site_rows(oracle, W.subject("optimized_transpose"), l)
    assert nv[0][3] == 4 and op[3][3] == 4
    assert nv[0][5] == op[3][5] == 16 * 2
