// device_rt.cuh — device runtime of the pgvc evaluation kernel (K2), sm_100a.
//
// Compiled by NVRTC together with the per-kernel code that codegen.cpp emits
// from the IR.  This file implements, for every emulated thread of every
// emulated block of every (launch, seed) instance packed into a CTA:
//   * round (barrier-interval) execution, PAPER.md L150-L152 / L658-L662,
//     with the write-log visibility rule X3 and min-tid commit X4;
//   * the write-ownership scatter: one 64-bit atomicMin of (stamp, value) per
//     logged write both selects the unique writer of the round (the fresh
//     writer thread of Fig. 2) and commits its value (H4/H5);
//   * WW / RW / XB race and OOB / UNINIT / LIMIT detection (X4-X6, X19);
//   * warp-level bank-conflict and coalescing measurement with
//     __match_any_sync / __ballot_sync / __reduce_*_sync (X9, H6);
//   * per-thread minimum events, flushed into the (instance, kernel, kind)
//     record slots (X16, H8).
// Nothing here knows the subject kernel: codegen.cpp supplies PG_* macros,
// the Frame struct and the segment function.
#pragma once

#include "pg_layout.h"

// ------------------------------------------------------------------ arithmetic (X2)
#define PG_MASK (PG_BITS >= 32 ? 0xFFFFFFFFu : ((1u << (PG_BITS & 31)) - 1u))
__device__ __forceinline__ u32 pg_m(u32 v) { return PG_BITS >= 32 ? v : (v & PG_MASK); }
__device__ __forceinline__ i32 pg_sx(u32 v) {
    if (PG_BITS >= 32) return (i32)v;
    return (i32)(v << (32 - PG_BITS)) >> (32 - PG_BITS);
}
__device__ __forceinline__ u32 pg_add(u32 a, u32 b) { return pg_m(a + b); }
__device__ __forceinline__ u32 pg_sub(u32 a, u32 b) { return pg_m(a - b); }
__device__ __forceinline__ u32 pg_mul(u32 a, u32 b) { return pg_m(a * b); }
__device__ __forceinline__ u32 pg_udiv(u32 a, u32 b) { return b ? a / b : PG_MASK; }
__device__ __forceinline__ u32 pg_urem(u32 a, u32 b) { return b ? a % b : a; }
__device__ __forceinline__ u32 pg_sdiv(u32 a, u32 b) {
    i32 x = pg_sx(a), y = pg_sx(b);
    if (y == 0) return x < 0 ? 1u : PG_MASK;
    if (y == -1) return pg_m(0u - (u32)x);  // INT_MIN / -1 wraps
    return pg_m((u32)(x / y));
}
__device__ __forceinline__ u32 pg_srem(u32 a, u32 b) {
    i32 x = pg_sx(a), y = pg_sx(b);
    if (y == 0) return a;
    if (y == -1) return 0u;
    return pg_m((u32)(x % y));
}
__device__ __forceinline__ u32 pg_shl(u32 a, u32 b) { return b >= (u32)PG_BITS ? 0u : pg_m(a << b); }
__device__ __forceinline__ u32 pg_lshr(u32 a, u32 b) { return b >= (u32)PG_BITS ? 0u : (a >> b); }
__device__ __forceinline__ u32 pg_ashr(u32 a, u32 b) {
    i32 x = pg_sx(a);
    if (b >= (u32)PG_BITS) return x < 0 ? PG_MASK : 0u;
    return pg_m((u32)(x >> b));
}
__device__ __forceinline__ u32 pg_slt(u32 a, u32 b) { return pg_sx(a) < pg_sx(b); }
__device__ __forceinline__ u32 pg_sle(u32 a, u32 b) { return pg_sx(a) <= pg_sx(b); }
__device__ __forceinline__ u32 pg_neg(u32 a) { return pg_m(0u - a); }
__device__ __forceinline__ u32 pg_not(u32 a) { return pg_m(~a); }

// ------------------------------------------------------------------ PRF (X8)
#include "pg_prf.cuh"

// ------------------------------------------------------------------ state
struct PgC {                 // CTA-uniform state
    const PgLaunchK* L;      // in shared memory
    u32 round;               // round index within the block (record field)
    u32 step;                // round index within the instance, 1-based (stamps)
    u32 fuel;
    u32 ufuel;               // uniform-loop iterations this round
};

struct PgT {                 // per emulated thread
    u32 live;                // 0/1: not exited and a real thread of a real instance
    u32 blk, bid[3];         // emulated block (linear id and bid.xyz)
    u32 tid[3];
    u32 tlin, gtid;
    u32 lane, ekey;          // HW lane; emulated-warp key within the HW warp (63: idle lane)
    u32 nlog;
    u32 fuel;
    u64 seed;
    u32* arena;              // this instance's kernel arena
    const u32* input;        // this instance's input region
    unsigned char* sgrp;     // this instance's shared-array region
    u32 lcell[PG_WMAX];      // write log (X3): cell id = array << 24 | flat
    u32 lval[PG_WMAX];
    u16 lsite[PG_WMAX];
    u32 ecnt[PG_NK];         // events per kind
    u32 ebest[PG_NK][8];     // minimum event per kind (X16)
};

__device__ __forceinline__ bool pg_lex_less(const u32* a, const u32* b) {
#pragma unroll
    for (int i = 0; i < 8; i++) {
        if (a[i] != b[i]) return a[i] < b[i];
    }
    return false;
}

__device__ __noinline__ void pg_event(PgT& t, u32 kind, u32 round, u32 arr, u32 addr, u32 ta, u32 tb, u32 site,
                                      u32 va, u32 vb) {
    u32 e[8] = {round, arr, addr, ta, tb, site, va, vb};
    if (t.ecnt[kind] == 0 || pg_lex_less(e, t.ebest[kind])) {
#pragma unroll
        for (int i = 0; i < 8; i++) t.ebest[kind][i] = e[i];
    }
    t.ecnt[kind]++;
}

// ------------------------------------------------------------------ array addressing
template <int A>
__device__ __forceinline__ const PgArr& pg_arr(const PgC& C) {
    return C.L->arr[A];
}
template <int A>
__device__ __forceinline__ u64* pg_sh_cells(const PgC& C, const PgT& t) {
    return (u64*)(t.sgrp + C.L->arr[A].smem_cells);
}
template <int A>
__device__ __forceinline__ u32* pg_sh_u32(const PgT& t, u32 off) {
    return (u32*)(t.sgrp + off);
}

// stamps: step (20 bits, >= 1) and block-local tid (12 bits)
__device__ __forceinline__ u32 pg_stamp_min(const PgC& C, const PgT& t) { return ((0xFFFFFu - C.step) << 12) | t.tlin; }
__device__ __forceinline__ u32 pg_stamp_max(const PgC& C, const PgT& t) { return (C.step << 12) | t.tlin; }

// ------------------------------------------------------------------ bank / coalescing (X9, H6)
#if PG_BANKCHK || PG_COALCHK
extern __shared__ __align__(16) unsigned char pg_dsmem[];
__device__ __forceinline__ void pg_site_stat(u64* st, u32 space, u32 bad, u32 metric, u32 ideal, u32 lanes) {
    // [space, n_acc, n_bad, max, sum, sum_ideal, sum_lanes, 0]
    st[0] = space;
    atomicAdd(&st[1], 1ull);
    if (bad) atomicAdd(&st[2], 1ull);
    atomicMax(&st[3], (u64)metric);
    atomicAdd(&st[4], (u64)metric);
    atomicAdd(&st[5], (u64)ideal);
    atomicAdd(&st[6], (u64)lanes);
}
#endif

// All 32 lanes of the warp call this together (the generated code keeps
// warps converged around every access site).
__device__ __noinline__ void pg_bank_shared(PgC& C, PgT& t, u64* sstats, u32 active, u32 rec, u32 flat, u32 site) {
#if PG_BANKCHK
    const u32 lane = t.lane;
    u32 ekey = t.ekey;
    if (PG_BANK16) ekey = ekey * 2u + ((t.tlin >> 4) & 1u);
    const u32 seg = __match_any_sync(PG_FULL, ekey);
    const u32 amask = __ballot_sync(PG_FULL, active) & seg;
    const u32 nb = PG_BANK16 ? 16u : 32u;
    const u32 bank = active ? flat % nb : 0u;
    const u32 w = active ? flat : 0u;
    const u32 mb = __match_any_sync(PG_FULL, (ekey << 7) | (active << 6) | bank);
    const u32 mw = __match_any_sync(PG_FULL, (ekey << 25) | (active << 24) | (w & 0xFFFFFFu));
    const u32 lead = __ballot_sync(PG_FULL, active && (u32)(__ffs(mw) - 1) == lane);
    const u32 mine = active ? (u32)__popc(mb & lead) : 0u;
    const u32 deg = __reduce_max_sync(seg, mine);
    const u32 bstar = __reduce_min_sync(seg, (active && mine == deg) ? bank : PG_NEVER);
    const u32 astar = __reduce_min_sync(seg, (active && bank == bstar) ? flat : PG_NEVER);
    const u32 ta = __reduce_min_sync(seg, (active && flat == astar) ? t.gtid : PG_NEVER);
    const u32 tb = __reduce_min_sync(seg, (active && bank == bstar && flat != astar) ? t.gtid : PG_NEVER);
    if (amask && lane == (u32)(__ffs(amask) - 1)) {
        if (sstats && site < PG_NSTATS) pg_site_stat(sstats + site * 8, 1, deg > 1, deg, 1, __popc(amask));
        if (deg > 1) pg_event(t, PGK_BANK, C.round, rec, astar, ta, tb, site, deg, 0);
    }
#endif
}

__device__ __noinline__ void pg_coal_global(PgC& C, PgT& t, u64* sstats, u32 active, u32 rec, u32 flat, u32 site) {
#if PG_COALCHK
    const u32 lane = t.lane;
    const u32 ekey = t.ekey;
    const u32 seg = __match_any_sync(PG_FULL, ekey);
    const u32 amask = __ballot_sync(PG_FULL, active) & seg;
    const u32 w = active ? flat : 0u;
    const u32 mw = __match_any_sync(PG_FULL, (ekey << 25) | (active << 24) | (w & 0xFFFFFFu));
    const u32 ms = __match_any_sync(PG_FULL, (ekey << 25) | (active << 24) | ((w >> 3) & 0xFFFFFFu));
    const u32 lw = __ballot_sync(PG_FULL, active && (u32)(__ffs(mw) - 1) == lane) & amask;
    const u32 ls = __ballot_sync(PG_FULL, active && (u32)(__ffs(ms) - 1) == lane) & amask;
    const u32 words = __popc(lw), sectors = __popc(ls);
    const u32 ideal = (words + 7u) / 8u;
    const u32 amin = __reduce_min_sync(seg, active ? flat : PG_NEVER);
    const u32 ta = __reduce_min_sync(seg, active ? t.gtid : PG_NEVER);
    const u32 tb = __reduce_max_sync(seg, active ? t.gtid : 0u);
    if (amask && lane == (u32)(__ffs(amask) - 1)) {
        if (sstats && site < PG_NSTATS) pg_site_stat(sstats + site * 8, 2, sectors > ideal, sectors, ideal, __popc(amask));
        if (sectors > ideal) pg_event(t, PGK_UNCOAL, C.round, rec, amin, ta, tb, site, sectors, ideal);
    }
#endif
}

// ------------------------------------------------------------------ loads / stores
// Shared array A: u64 cells (stamp << 32 | value) in the group's region.
template <int A, bool RD>
__device__ __forceinline__ u32 pg_ld_sh(PgC& C, PgT& t, u64* ss, u32 pe, u32 flat, u32 site) {
    const PgArr& a = C.L->arr[A];
    const u32 inb = flat < a.size;
#if PG_BANKCHK
    pg_bank_shared(C, t, ss, pe & inb, a.rec_id, flat, site);
#endif
    if (!pe) return 0u;
    if (!inb) {
        u32 pv = pg_m(pg_rand32(t.seed, 0x8000u + (a.rec_id - 0x100u), ((u64)t.blk << 20) + flat));
#if PG_OOBCHK
        pg_event(t, PGK_OOB, C.round, a.rec_id, flat, t.gtid, PG_NEVER, site, pv, 0);
#endif
        return pv;
    }
#if PG_RACECHK
    if (RD) {
        atomicMin((u32*)(t.sgrp + a.smem_rmin) + flat, pg_stamp_min(C, t));
        atomicMax((u32*)(t.sgrp + a.smem_rmax) + flat, pg_stamp_max(C, t));
    }
#endif
    const u32 cell = ((u32)A << 24) | flat;
    for (u32 i = 0; i < t.nlog; i++)
        if (t.lcell[i] == cell) return t.lval[i];
    const u64 c = ((const u64*)(t.sgrp + a.smem_cells))[flat];
    if ((u32)(c >> 32) == PG_NEVER) {
        u32 pv = pg_m(pg_rand32(t.seed, 0x8000u + (a.rec_id - 0x100u), ((u64)t.blk << 20) + flat));
#if PG_OOBCHK
        pg_event(t, PGK_UNINIT, C.round, a.rec_id, flat, t.gtid, PG_NEVER, site, pv, 0);
#endif
        return pv;
    }
    return (u32)c;
}

__device__ __noinline__ void pg_log_write(PgC& C, PgT& t, u32 cell, u32 val, u32 site, u32 rec, u32 flat) {
    for (u32 i = 0; i < t.nlog; i++) {
        if (t.lcell[i] == cell) {
            t.lval[i] = val;
            t.lsite[i] = (u16)site;
            return;
        }
    }
    if (t.nlog >= PG_WMAX) {  // X19: write-log limit, the write is dropped
        pg_event(t, PGK_LIMIT, C.round, rec, flat, t.gtid, PG_NEVER, site, 1, 0);
        return;
    }
    t.lcell[t.nlog] = cell;
    t.lval[t.nlog] = val;
    t.lsite[t.nlog] = (u16)site;
    t.nlog++;
}

template <int A>
__device__ __forceinline__ void pg_st_sh(PgC& C, PgT& t, u64* ss, u32 pe, u32 flat, u32 val, u32 site) {
    const PgArr& a = C.L->arr[A];
    const u32 inb = flat < a.size;
#if PG_BANKCHK
    pg_bank_shared(C, t, ss, pe & inb, a.rec_id, flat, site);
#endif
    if (!pe) return;
    if (!inb) {
#if PG_OOBCHK
        pg_event(t, PGK_OOB, C.round, a.rec_id, flat, t.gtid, PG_NEVER, site, val, 1);
#endif
        return;
    }
    pg_log_write(C, t, ((u32)A << 24) | flat, val, site, a.rec_id, flat);
}

// Global array written by this kernel: u64 cells in the instance arena.
// XB bookkeeping (X4): first and last block that accessed a global cell.  Kept
// whenever the launch has more than one block (it also decides whether the
// block-parallel pass must be redone sequentially).
template <int A>
__device__ __forceinline__ void pg_xb_mark(const PgC& C, PgT& t, const PgArr& a, u32 flat) {
    if (a.off_xf != ~0ull) {
        atomicMin(t.arena + a.off_xf + flat, t.blk + 1u);
        atomicMax(t.arena + a.off_xl + flat, t.blk + 1u);
    }
}

template <int A, bool RD>
__device__ __forceinline__ u32 pg_ld_gt(PgC& C, PgT& t, u64* ss, u32 pe, u32 flat, u32 site) {
    const PgArr& a = C.L->arr[A];
    const u32 inb = flat < a.size;
#if PG_COALCHK
    pg_coal_global(C, t, ss, pe & inb, a.rec_id, flat, site);
#endif
    if (!pe) return 0u;
    if (!inb) {
        u32 pv = pg_m(pg_rand32(t.seed, a.gid, flat));
#if PG_OOBCHK
        pg_event(t, PGK_OOB, C.round, a.rec_id, flat, t.gtid, PG_NEVER, site, pv, 0);
#endif
        return pv;
    }
    pg_xb_mark<A>(C, t, a, flat);
#if PG_RACECHK
    if (RD) {
        atomicMin(t.arena + a.off_rmin + flat, pg_stamp_min(C, t));
        atomicMax(t.arena + a.off_rmax + flat, pg_stamp_max(C, t));
    }
#endif
    const u32 cell = ((u32)A << 24) | flat;
    for (u32 i = 0; i < t.nlog; i++)
        if (t.lcell[i] == cell) return t.lval[i];
    return (u32)((const u64*)(t.arena + a.off_cells))[flat];
}

template <int A>
__device__ __forceinline__ void pg_st_gt(PgC& C, PgT& t, u64* ss, u32 pe, u32 flat, u32 val, u32 site) {
    const PgArr& a = C.L->arr[A];
    const u32 inb = flat < a.size;
#if PG_COALCHK
    pg_coal_global(C, t, ss, pe & inb, a.rec_id, flat, site);
#endif
    if (!pe) return;
    if (!inb) {
#if PG_OOBCHK
        pg_event(t, PGK_OOB, C.round, a.rec_id, flat, t.gtid, PG_NEVER, site, val, 1);
#endif
        return;
    }
    pg_xb_mark<A>(C, t, a, flat);
    pg_log_write(C, t, ((u32)A << 24) | flat, val, site, a.rec_id, flat);
}

// Global array this kernel only reads: the instance's input region.
template <int A>
__device__ __forceinline__ u32 pg_ld_gi(PgC& C, PgT& t, u64* ss, u32 pe, u32 flat, u32 site) {
    const PgArr& a = C.L->arr[A];
    const u32 inb = flat < a.size;
#if PG_COALCHK
    pg_coal_global(C, t, ss, pe & inb, a.rec_id, flat, site);
#endif
    if (!pe) return 0u;
    if (!inb) {
        u32 pv = pg_m(pg_rand32(t.seed, a.gid, flat));
#if PG_OOBCHK
        pg_event(t, PGK_OOB, C.round, a.rec_id, flat, t.gtid, PG_NEVER, site, pv, 0);
#endif
        return pv;
    }
    return __ldg(t.input + a.off_in + flat);
}

// Private (per-thread) array: bounds check only (X5); no races, no logging.
__device__ __forceinline__ u32 pg_priv_ok(PgC& C, PgT& t, u32 pe, u32 flat, u32 size, u32 rec, u32 site, u32 val,
                                          u32 is_store) {
    if (!pe) return 0u;
    if (flat < size) return 1u;
#if PG_OOBCHK
    pg_event(t, PGK_OOB, C.round, rec, flat, t.gtid, PG_NEVER, site, is_store ? val : 0u, is_store);
#endif
    return 0u;
}

// ------------------------------------------------------------------ loops (fuel, X19)
__device__ __forceinline__ void pg_tick(PgC& C, PgT& t, u32 act) {
    if (act && ++t.fuel > C.fuel) {
        pg_event(t, PGK_LIMIT, C.round, PG_NEVER, 0, t.gtid, PG_NEVER, PG_NEVER, 2, 0);
        t.live = 0;
    }
}

// ------------------------------------------------------------------ round end (H4)
// Phase 1 (claim/commit): each logged write does atomicMin on its cell with
// (stamp_min << 32 | value): the newest round wins over stale stamps, the
// min tid wins within the round, and the winner's value is committed by the
// same atomic.  Phase 2 (check): the owner of a global cell records itself as
// the last writer; with race checks, WW is reported by the max-tid writer and
// RW by the thread named tid_a by the X16 rule.
__device__ __forceinline__ u64* pg_cell_ptr(const PgC& C, const PgT& t, u32 a, u32 flat) {
    const PgArr& ar = C.L->arr[a];
    if (ar.kind == PGA_SH) return (u64*)(t.sgrp + ar.smem_cells) + flat;
    return (u64*)(t.arena + ar.off_cells) + flat;
}
__device__ __forceinline__ u32* pg_stamp_ptr(const PgT& t, const PgArr& ar, u32 smem_off, u64 gl_off) {
    return ar.kind == PGA_SH ? (u32*)(t.sgrp + smem_off) : t.arena + gl_off;
}

__device__ __noinline__ void pg_claim(const PgC& C, PgT& t) {
    const u32 smin = pg_stamp_min(C, t);
    for (u32 i = 0; i < t.nlog; i++) {
        const u32 a = t.lcell[i] >> 24, flat = t.lcell[i] & 0xFFFFFFu;
        atomicMin(pg_cell_ptr(C, t, a, flat), ((u64)smin << 32) | t.lval[i]);
#if PG_RACECHK
        const PgArr& ar = C.L->arr[a];
        atomicMax(pg_stamp_ptr(t, ar, ar.smem_wmax, ar.off_wmax) + flat, pg_stamp_max(C, t));
#endif
    }
}

__device__ __noinline__ void pg_check(const PgC& C, PgT& t) {
    const u32 smin = pg_stamp_min(C, t);
    const u32 base = t.gtid - t.tlin;
    for (u32 i = 0; i < t.nlog; i++) {
        const u32 a = t.lcell[i] >> 24, flat = t.lcell[i] & 0xFFFFFFu;
        const PgArr& ar = C.L->arr[a];
        const u64 c = *pg_cell_ptr(C, t, a, flat);
        const u32 owner_stamp = (u32)(c >> 32);
        if (ar.kind == PGA_GT && owner_stamp == smin) t.arena[ar.off_lw + flat] = t.gtid + 1u;
#if PG_RACECHK
        const u32 w0 = owner_stamp & 0xFFFu;
        const u32 w1 = pg_stamp_ptr(t, ar, ar.smem_wmax, ar.off_wmax)[flat] & 0xFFFu;
        if (w1 != w0 && t.tlin == w1)
            pg_event(t, PGK_WW, C.round, ar.rec_id, flat, base + w0, t.gtid, t.lsite[i], (u32)c, t.lval[i]);
        if (ar.flags & 1u) {
            const u32 rmx = pg_stamp_ptr(t, ar, ar.smem_rmax, ar.off_rmax)[flat];
            if ((rmx >> 12) == C.step) {
                const u32 r0 = pg_stamp_ptr(t, ar, ar.smem_rmin, ar.off_rmin)[flat] & 0xFFFu, r1 = rmx & 0xFFFu;
                if (!(r0 == r1 && w0 == w1 && r0 == w0)) {
                    u32 ta, tb;
                    if (r0 != w0) { ta = w0; tb = r0; }
                    else if (r1 != w0) { ta = w0; tb = r1; }
                    else { ta = w1; tb = r0; }
                    if (t.tlin == ta)
                        pg_event(t, PGK_RW, C.round, ar.rec_id, flat, base + ta, base + tb, t.lsite[i], t.lval[i], 0);
                }
            }
        }
#endif
    }
}

// ------------------------------------------------------------------ records (H8)
// Each thread keeps its minimum event per kind; at the end of the CTA the lanes
// of a warp that belong to the same instance merge theirs (lexicographic min by
// successive warp-wide minima, counts by warp sum) and one lane updates the
// (instance, kernel, kind) slot under its lock.  All 32 lanes call this.
__device__ __noinline__ void pg_flush_warp(const PgParams& P, PgT& t, u32 valid, u64 slot0) {
    for (u32 k = 0; k < PG_NK; k++) {
        u32 pending = valid && t.ecnt[k] != 0u;
        for (;;) {
            const u32 pm = __ballot_sync(PG_FULL, pending);
            if (!pm) break;
            const u32 leader = (u32)__ffs(pm) - 1u;
            const u64 lslot = __shfl_sync(PG_FULL, slot0, leader);
            u32 cand = pending && slot0 == lslot;
            const u32 members = __ballot_sync(PG_FULL, cand);
            const u32 cnt = __reduce_add_sync(PG_FULL, cand ? t.ecnt[k] : 0u);
            u32 best[8];
#pragma unroll
            for (int f = 0; f < 8; f++) {
                best[f] = __reduce_min_sync(PG_FULL, cand ? t.ebest[k][f] : PG_NEVER);
                cand = cand && t.ebest[k][f] == best[f];
            }
            if (t.lane == leader) {
                PgSlot* s = P.slots + lslot + k;
                atomicAdd(&s->count, (u64)cnt);
                while (atomicCAS(&s->lock, 0u, 1u) != 0u) {
                }
                __threadfence();
                volatile PgSlot* vs = s;
                u32 cur[8];
#pragma unroll
                for (int i = 0; i < 8; i++) cur[i] = vs->f[i];
                if (!vs->has || pg_lex_less(best, cur)) {
#pragma unroll
                    for (int i = 0; i < 8; i++) vs->f[i] = best[i];
                    vs->has = 1u;
                }
                __threadfence();
                atomicExch(&s->lock, 0u);
            }
            if (members & (1u << t.lane)) pending = 0u;
            __syncwarp();
        }
    }
}

// ------------------------------------------------------------------ CTA main loop
// A CTA runs P groups of one launch in lock step.  Group g emulates, for seed
// (g / gb) of the work item, the blocks blk0 + i*gb + (g % gb), i = 0, 1, ...
// (gb > 1 only when no block-uniform branch depends on bid, so all groups share
// one round structure).  Blocks of one instance therefore run in parallel
// (across groups and CTAs); that is exact unless a global cell is shared
// between blocks (XB), which K2b detects - those seed groups are re-run by the
// sequential pass (P.seq = 1: gb = 1, all blocks in linear bid order, X21).
#ifndef PG_VMAX
#define PG_VMAX 1
#endif

__device__ __forceinline__ u32 pg_init_value(const PgParams& P, u64 seed, u32 gid, u32 i) {
    u32 v;
    if (P.input_mode == 1) v = i < 64 ? (u32)((seed >> i) & 1ull) : 0u;
    else if (P.input_mode == 2) v = pg_rand32(seed, gid, i) % (P.input_range ? P.input_range : 1u);
    else v = pg_rand32(seed, gid, i);
    return v & P.mask;
}

template <class K>
__device__ __forceinline__ void pg_main(const PgParams& P) {
    extern __shared__ __align__(16) unsigned char pg_dsmem[];
    __shared__ PgLaunchK sL;
    __shared__ PgWork sW;
    __shared__ u32 s_flag;
    {
        const u32* src = (const u32*)&P.launches[P.work[blockIdx.x].launch];
        u32* dst = (u32*)&sL;
        for (u32 i = threadIdx.x; i < sizeof(PgLaunchK) / 4; i += blockDim.x) dst[i] = src[i];
        const u32* ws = (const u32*)&P.work[blockIdx.x];
        u32* wd = (u32*)&sW;
        for (u32 i = threadIdx.x; i < sizeof(PgWork) / 4; i += blockDim.x) wd[i] = ws[i];
    }
    __syncthreads();
    const PgLaunchK& L = sL;
    const u32 G = sW.ngroups, GB = sW.gb;
    if (P.seq) {
        // re-run only seed groups in which some instance shared a global cell between blocks
        if (threadIdx.x == 0) {
            u32 f = 0;
            for (u32 i = 0; i < sW.nseeds; i++) f |= P.xb_flag[sW.inst0 + i];
            s_flag = f;
        }
        __syncthreads();
        if (!s_flag) return;
        // fresh arenas and slots for every seed of the group (the parallel pass is discarded)
        for (u32 ms = 0; ms < sW.nseeds; ms++) {
            const u64 seed = P.seed_base + (u64)(sW.seed_j0 + ms * sW.seed_jstep);
            u32* ar = P.arena + sW.arena_off + (u64)ms * L.arena_stride;
            for (u32 a = 0; a < L.n_arrays; a++) {
                const PgArr& R = L.arr[a];
                if (R.kind != PGA_GT) continue;
                u64* cells = (u64*)(ar + R.off_cells);
                for (u32 i = threadIdx.x; i < R.size; i += blockDim.x) {
                    cells[i] = ((u64)PG_NEVER << 32) | pg_init_value(P, seed, R.gid, i);
                    ar[R.off_lw + i] = 0u;
                    if (R.off_wmax != ~0ull) ar[R.off_wmax + i] = 0u;
                    if (R.off_rmin != ~0ull) ar[R.off_rmin + i] = PG_NEVER;
                    if (R.off_rmax != ~0ull) ar[R.off_rmax + i] = 0u;
                    if (R.off_xf != ~0ull) { ar[R.off_xf + i] = PG_NEVER; ar[R.off_xl + i] = 0u; }
                }
            }
            if (threadIdx.x < PG_NK) {
                PgSlot* sl = P.slots + sW.slot0 + (u64)ms * sW.slot_step + threadIdx.x;
                sl->count = 0;
                sl->has = 0;
                sl->lock = 0;
            }
        }
        __threadfence();
        __syncthreads();
    }
    unsigned char* sgroups = pg_dsmem;
    u64* sstats = (u64*)(pg_dsmem + (u64)L.P * L.smem_group_bytes);
    u32* s_alive = (u32*)(sstats + ((PG_BANKCHK || PG_COALCHK) ? PG_NSTATS * 8 : 0));
    u32* s_alive_next = s_alive + L.P;
    u32* s_rounds = s_alive_next + L.P;
    u64* s_inst = (u64*)(((unsigned long long)(s_rounds + L.P) + 7) & ~7ull);
#if PG_BANKCHK || PG_COALCHK
    for (u32 i = threadIdx.x; i < PG_NSTATS * 8; i += blockDim.x) sstats[i] = 0;
#else
    sstats = nullptr;
#endif
    for (u32 i = threadIdx.x; i < L.P; i += blockDim.x) { s_inst[i] = 0; s_alive_next[i] = 0; }

    PgC C;
    C.L = &sL;
    C.step = 0;
    C.fuel = P.fuel;
    const u32 lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    u32 g, tl0, lane_ok, ekey;
    if (L.T <= 32u) {
        const u32 sub = lane / L.T;
        g = warp * L.gpw + sub;
        tl0 = lane - sub * L.T;
        lane_ok = sub < L.gpw;
        ekey = lane_ok ? sub : 63u;
    } else {
        g = warp / L.wpg;
        tl0 = (warp % L.wpg) * 32u + lane;
        lane_ok = 1u;
        ekey = 0u;
    }
    const u32 inst_ok = lane_ok && g < G;
    const u32 gc = inst_ok ? g : 0u;
    const u32 ms = gc / GB, bs = gc % GB;
    typename K::Frame F[PG_VMAX];
    PgT T[PG_VMAX];
    const u32 V = PG_VMAX > 1 ? L.V : 1u;
#pragma unroll
    for (u32 v = 0; v < PG_VMAX; v++) {
        if (v >= V) break;
        PgT& t = T[v];
        t.tlin = tl0 + v * 1024u;
        const u32 ok = inst_ok && t.tlin < L.T;
        t.ekey = ok ? ekey : 63u;
        t.lane = lane;
        t.tid[0] = t.tlin % L.bdim[0];
        t.tid[1] = (t.tlin / L.bdim[0]) % L.bdim[1];
        t.tid[2] = t.tlin / (L.bdim[0] * L.bdim[1]);
        t.seed = P.seed_base + (u64)(sW.seed_j0 + ms * sW.seed_jstep);
        t.arena = P.arena + sW.arena_off + (u64)ms * L.arena_stride;
        t.input = P.input + sW.input_off + (u64)ms * L.input_stride;
        t.sgrp = sgroups + (u64)gc * L.smem_group_bytes;
        for (u32 k = 0; k < PG_NK; k++) t.ecnt[k] = 0;
        t.live = ok;
    }
    const u32 nsteps = (sW.blk1 - sW.blk0 + GB - 1) / GB;
    for (u32 st = 0; st < nsteps; st++) {
        const u32 blk = sW.blk0 + st * GB + bs;
        const u32 blk_ok = blk < sW.blk1;
        // fresh shared arrays for every group: cells never written, stamps cleared
        {
            const u32 cw = L.smem_cells_bytes / 8u;
            const u32 zw = (L.smem_never_off - L.smem_cells_bytes) / 4u;
            const u32 nw = (L.smem_group_bytes - L.smem_never_off) / 4u;
            for (u32 gi = 0; gi < G; gi++) {
                unsigned char* base = sgroups + (u64)gi * L.smem_group_bytes;
                u64* cells = (u64*)base;
                for (u32 i = threadIdx.x; i < cw; i += blockDim.x) cells[i] = ((u64)PG_NEVER) << 32;
                u32* z = (u32*)(base + L.smem_cells_bytes);
                for (u32 i = threadIdx.x; i < zw; i += blockDim.x) z[i] = 0u;
                u32* nv = (u32*)(base + L.smem_never_off);
                for (u32 i = threadIdx.x; i < nw; i += blockDim.x) nv[i] = PG_NEVER;
            }
        }
        for (u32 i = threadIdx.x; i < L.P; i += blockDim.x) {
            s_alive[i] = i < G && sW.blk0 + st * GB + (i % GB) < sW.blk1;
            s_rounds[i] = 0;
        }
        __syncthreads();
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++) {
            if (v >= V) break;
            PgT& t = T[v];
            t.blk = blk;
            t.bid[0] = blk % L.gdim[0];
            t.bid[1] = (blk / L.gdim[0]) % L.gdim[1];
            t.bid[2] = blk / (L.gdim[0] * L.gdim[1]);
            t.live = inst_ok && t.tlin < L.T && blk_ok;
            t.gtid = blk * L.T + t.tlin;
            K::init(F[v], C, t);
        }
        C.round = 0;
        u32 resume = 0;
        for (;;) {
            C.step++;
            C.ufuel = 0;
            u32 r = PG_END;
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                T[v].nlog = 0;
                T[v].fuel = 0;
                r = K::seg(F[v], C, T[v], sstats, resume);
            }
            __syncthreads();
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                pg_claim(C, T[v]);
            }
            __syncthreads();
            u32 any = 0;
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                pg_check(C, T[v]);
                any |= T[v].live;
            }
            if (any && inst_ok) s_alive_next[g] = 1u;
            __syncthreads();
            for (u32 i = threadIdx.x; i < G; i += blockDim.x) {
                s_rounds[i] += s_alive[i];
                s_alive[i] = s_alive_next[i];
                s_alive_next[i] = 0u;
            }
            C.round++;
            const int more = __syncthreads_or((int)any);
            if (r == PG_END || !more) break;
            resume = r;
        }
        for (u32 i = threadIdx.x; i < G; i += blockDim.x) s_inst[i] += (u64)L.T * s_rounds[i];
        __syncthreads();
    }
#if PG_RACECHK
    // X4: cross-block races on global cells written by this kernel (sequential pass: the
    // CTA owns whole instances; the parallel pass leaves them to the flagged re-run)
    if (P.seq && L.nblocks > 1) {
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++) {
            if (v >= V) break;
            PgT& t = T[v];
            if (!(inst_ok && t.tlin < L.T)) continue;
            for (u32 a = 0; a < L.n_arrays; a++) {
                const PgArr& ar = L.arr[a];
                if (ar.kind != PGA_GT || ar.off_xf == ~0ull) continue;
                const u32* xf = t.arena + ar.off_xf;
                const u32* xl = t.arena + ar.off_xl;
                const u32* lw = t.arena + ar.off_lw;
                const u64* cells = (const u64*)(t.arena + ar.off_cells);
                for (u32 i = t.tlin; i < ar.size; i += L.T)
                    if (lw[i] && xf[i] != xl[i])
                        pg_event(t, PGK_XB, 0xFFFFu, ar.rec_id, i, xf[i] - 1u, xl[i] - 1u, PG_NEVER, (u32)cells[i], 0u);
            }
        }
    }
#endif
#pragma unroll
    for (u32 v = 0; v < PG_VMAX; v++) {
        if (v >= V) break;
        pg_flush_warp(P, T[v], inst_ok && T[v].tlin < L.T, sW.slot0 + (u64)ms * sW.slot_step);
    }
    if (!P.seq && inst_ok && tl0 == 0u) atomicAdd(&P.counts[0], s_inst[g]);
#if PG_BANKCHK || PG_COALCHK
    __syncthreads();
    if (P.site_stats) {
        u64* dst = P.site_stats + (u64)(P.seq ? sW.launch : sW.item) * P.max_sites * 8u;
        for (u32 i = threadIdx.x; i < PG_NSTATS * 8 && i < P.max_sites * 8; i += blockDim.x) {
            const u32 c = i & 7u;
            if (c == 3) atomicMax(&dst[i], sstats[i]);
            else if (c == 0) { if (sstats[i]) dst[i] = sstats[i]; }
            else if (sstats[i]) atomicAdd(&dst[i], sstats[i]);
        }
    }
#endif
}
