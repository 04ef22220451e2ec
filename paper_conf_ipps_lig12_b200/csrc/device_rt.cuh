// device_rt.cuh — device runtime of the pgvc evaluation kernel (K2), sm_100a.
//
// Compiled by NVRTC together with the per-kernel code that codegen.cpp emits
// from the IR.  It implements, for every emulated thread of every emulated
// block of every (launch, seed) instance packed into a CTA:
//   * round (barrier-interval) execution, PAPER.md L150-L152 / L658-L662,
//     with the write-log visibility rule X3 and the min-tid commit of X4;
//   * the write-ownership scatter (H4/H5): one 32-bit atomicMin per logged
//     write on the cell's owner stamp ((2^20-1 - step) << 12 | tid) selects
//     the unique writer of the round - the fresh writer thread of Fig. 2
//     (L582-L599) - which then commits its value;
//   * WW / RW / XB race and OOB / UNINIT / LIMIT detection (X4-X6, X19);
//   * warp-level bank-conflict and coalescing measurement with
//     __match_any_sync / __ballot_sync / __reduce_*_sync (X9, H6);
//   * per-thread minimum events, merged per warp and flushed into the
//     (instance, kernel, kind) record slots (X16, H8).
// Stamps carry the round step, so nothing is cleared between emulated blocks:
// a stamp older than the current block reads as "never written".
// codegen.cpp supplies the PG_* macros, the Frame struct, the segment function
// and the per-array claim/check dispatch.
#pragma once

#include "pg_layout.h"

// multi-seed lanes: PG_MS seeds per lane; PG_MSX: the exact protocol's
// multi-seed variant (the re-run of instances the multi-seed optimistic pass flagged)
#ifndef PG_MS
#define PG_MS 1
#endif
#ifndef PG_FAST
#define PG_FAST 0
#endif
#ifndef PG_OPCOUNT
#define PG_OPCOUNT 0   // PG_CHK_OPCOUNT: count executed IR operations (measurement variant)
#endif
#ifndef PG_DIVBAR
#define PG_DIVBAR 0    // a barrier under thread-dependent control: per-thread resume points (X18)
#endif
#ifndef PG_VCLIT
#define PG_VCLIT 0
#endif
// the exact protocol claims a cell when the store enters the write log (the claim words are
// separate from the committed-owner words loads consult), so a round needs two barriers, not
// three; the diagnostic variants (data-flow dump, VC-literal, lock-step) and run-time barrier
// divergence keep the separate claim phase
#ifndef PG_CAS_ON
#define PG_CAS_ON 1    // (PGVC_CAS=0: claims in their own phase, diagnostics)
#endif
// the round-end race decision of a racy cell (cold: one thread per racy cell and round)
#ifndef PG_RC_INLINE
#define PG_RC_INLINE __noinline__
#endif
#define PG_CAS (PG_CAS_ON && !PG_FAST && !PG_DATAFLOW && !PG_VCLIT && !PG_DIVBAR && !PG_LOCKSTEP)
#define PG_MSX (PG_MS > 1 && !PG_FAST)
#define PG_S_LOOP _Pragma("unroll") for (u32 _s = 0; _s < (u32)PG_MS; _s++)

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
// power-of-two divisors (e.g. the SDK reductions' 2*s) take the shift/mask identity
__device__ __forceinline__ u32 pg_udiv(u32 a, u32 b) {
    if (b && !(b & (b - 1u))) return a >> (__ffs(b) - 1);
    return b ? a / b : PG_MASK;
}
__device__ __forceinline__ u32 pg_urem(u32 a, u32 b) {
    if (b && !(b & (b - 1u))) return a & (b - 1u);
    return b ? a % b : a;
}
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
extern __shared__ __align__(16) unsigned char pg_dsmem[];  // group regions | site stats | group counters
__shared__ __align__(16) PgLaunchK pg_sL;                   // this CTA's launch descriptor (TMA bulk copy)
__shared__ __align__(8) u64 pg_sBar;                        // its mbarrier (complete_tx of the bulk copy)
__shared__ PgWork pg_sW;                                    // this CTA's work item

#define PG_ARR(A) (pg_sL.arr[A])
#define PG_LOCK_R 32u   // = PG_LOCK_ROUNDS (include/pgvc.h)

// Launch-shape constants.  A variant compiled for one block shape (api.cpp,
// shape_prelude) defines PG_S_*, and PgSA<A> for the shared-array layout: block
// size, shared offsets and CTA packing become immediates.  Otherwise they are read
// from the CTA's launch descriptor.
#ifdef PG_S_T
#define PG_T ((u32)PG_S_T)
#define PG_BDIM0 ((u32)PG_S_B0)
#define PG_BDIM1 ((u32)PG_S_B1)
#define PG_BDIM2 ((u32)PG_S_B2)
#define PG_SH(A, f) ((u32)PgSA<A>::f)
#define PG_GBYTES ((u32)PG_S_GBYTES)
#define PG_ZOFF ((u32)PG_S_ZOFF)
#define PG_NOFF ((u32)PG_S_NOFF)
#define PG_GPW ((u32)PG_S_GPW)
#define PG_WPG ((u32)PG_S_WPG)
#define PG_PK ((u32)PG_S_P)
#define PG_VV ((u32)PG_S_V)
#else
#define PG_T (pg_sL.T)
#define PG_BDIM0 (pg_sL.bdim[0])
#define PG_BDIM1 (pg_sL.bdim[1])
#define PG_BDIM2 (pg_sL.bdim[2])
#define PG_SH(A, f) (pg_sL.arr[A].f)
#define PG_GBYTES (pg_sL.smem_group_bytes)
#define PG_ZOFF (pg_sL.smem_zero_off)
#define PG_NOFF (pg_sL.smem_never_off)
#define PG_GPW (pg_sL.gpw)
#define PG_WPG (pg_sL.wpg)
#define PG_PK (pg_sL.P)
#define PG_VV (pg_sL.V)
#endif

struct PgC {        // CTA-uniform state
    u32 round;      // round index within the block (record field)
    u32 step;       // round counter of this CTA, >= 1 (stamps)
    u32 step0;      // step of the first round of the current block
    u32 fuel;
    u32 ufuel;      // uniform-loop iterations this round
    u32 abort;      // PG_FAST: a race was flagged, the item stops (its instances are re-run exactly)
    // derived from step / step0 once per round / block (pg_set_step, pg_set_step0)
    u32 smin;       // (2^20-1 - step) << 12: owner / min-reader stamp of this round without the tid
    u32 smax;       // step << 12: max-reader / max-writer stamp without the tid
    u32 par;        // step & 1: reader-stamp set of the optimistic pass
    u32 uthr;       // owner stamps >= uthr predate this block ("never written", X6)
};
__device__ __forceinline__ void pg_set_step(PgC& C, u32 s) {
    C.step = s;
    C.smin = (0xFFFFFu - s) << 12;
    C.smax = s << 12;
    C.par = s & 1u;
}
__device__ __forceinline__ void pg_set_step0(PgC& C, u32 s0) {
    C.step0 = s0;
    C.uthr = (0x100000u - s0) << 12;
}

struct PgT {        // hot per-emulated-thread state (kept in registers)
    u32 live;       // 0/1: not exited, and a real thread of a real instance and block
    u32 blk, bid[3];
    u32 tid[3];
    u32 tlin, gtid;
    u32 lane, ekey; // HW lane; emulated-warp key within the HW warp (63: idle)
    u32 nlog;
    u32 evm;        // kinds with a recorded event (bit k: PgCold::ecnt[k] / ebest[k] are valid)
    u32 fl;         // PG_FAST: this thread saw a possible race / write-log overflow (instance re-run exactly)
    u32 l0cell, l0val, l0site;  // write-log entry 0 (registers; entries 1.. live in PgCold)
#if PG_MSX
    u32 l0v[PG_MS];             // (multi-seed exact pass: entry 0's value per seed)
#endif
    u32 fuel;
    u32 sg;         // byte offset of this instance's shared region in pg_dsmem
    u32 nsv;        // multi-seed lanes: seeds of this lane's group (<= PG_MS)
#if PG_OPCOUNT
    u32 ops;        // IR integer operations this thread executed (PG_CHK_OPCOUNT)
#endif
    u64 seed;
    u32* arena;     // this instance's kernel arena
    const u32* input;
};

#if PG_MSX
typedef const u32* pg_lv_t;   // a write-log value: one word per seed
#else
typedef u32 pg_lv_t;
#endif
struct PgCold {     // per-emulated-thread state that lives in local memory
    u32 lcell[PG_WMAX];   // write log entries 1.. (X3): cell id = array << 24 | flat
    u32 lval[PG_WMAX];
    u16 lsite[PG_WMAX];
    u32 ecnt[PG_NK];      // events per kind       (valid where PgT::evm has bit k: never initialised,
    u32 ebest[PG_NK][8];  // minimum event per kind  so threads without events touch no local memory) (X16)
#if PG_MSX
    u32 lvs[PG_WMAX][PG_MS];   // (see pg_lv_t)     // write-log values per seed (entries 1..)
    u32 ebv[PG_NK][PG_MS];       // per seed: val_a of the minimum event; fields 0..5 of ebest are
                                 // seed-independent (same accesses in every seed)
    u32 ebvb[PG_NK];             // its val_b, which every event kind takes seed-independently (site,
                                 // degree, ...), so one word per kind (local-memory footprint) ...
    u32 vbx;                     // ... unless two events with equal fields 0..5 but different val_b
    u32 ebvs[PG_NK][PG_MS];      //     met (bit k): then val_b per seed here
#endif
    u64 epk[PG_NK];              // pg_pack of ebest[kind] (one 64-bit compare decides most events)
};

__device__ __forceinline__ bool pg_lex_less(const u32* a, const u32* b) {
#pragma unroll
    for (int i = 0; i < 8; i++) {
        if (a[i] != b[i]) return a[i] < b[i];
    }
    return false;
}

// Monotone 64-bit prefix of the X16 event order: (round, array, addr, tid_a) in 16 / 10 / 24 /
// 14 bits (in-bounds addresses are < 2^24, X5; tid_a is a global thread id, so the wider
// field separates the events of more blocks before the lexicographic fallback), a field
// that does not fit saturates and zeroes the rest, so a <lex b implies
// pg_pack(a) <= pg_pack(b).  Slots keep ~pg_pack of their minimum (atomicMax): a candidate
// whose pack is larger cannot be the minimum and skips the lock - thousands of CTAs that
// report events of one instance (one slot) no longer serialise on it.
#ifndef PG_PACK_B2
#define PG_PACK_B0 16u
#define PG_PACK_B1 10u
#define PG_PACK_B2 24u
#define PG_PACK_B3 14u
#endif
__device__ __forceinline__ u64 pg_pack(const u32* f) {
    const u32 bits[4] = {PG_PACK_B0, PG_PACK_B1, PG_PACK_B2, PG_PACK_B3};
    u64 k = 0;
    bool sat = false;
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const u64 mx = (1ull << bits[i]) - 1ull;
        u64 v = f[i];
        if (sat) v = 0;
        else if (v >= mx) { v = mx; sat = true; }
        k = (k << bits[i]) | v;
    }
    return k;
}
// Records an event of `kind`; `evm` is the caller's event mask (PgT::evm).  Returns the
// kind's bit, which the caller ORs into its mask.
// The packed prefix pg_pack of the kind's minimum (epk) decides most comparisons with one
// 64-bit load: a thread's events mostly arrive in increasing order (round first).
__device__ __noinline__ u32 pg_event(PgCold& c, u32 evm, u32 kind, u32 round, u32 arr, u32 addr, u32 ta, u32 tb,
                                     u32 site, u32 va, u32 vb) {
    u32 e[8] = {round, arr, addr, ta, tb, site, va, vb};
    const u32 has = (evm >> kind) & 1u;
    const u64 pk = pg_pack(e);
    bool take = !has;
    if (has) {
        const u64 bp = c.epk[kind];
        take = pk < bp || (pk == bp && pg_lex_less(e, c.ebest[kind]));
    }
    if (take) {
        c.epk[kind] = pk;
#pragma unroll
        for (int i = 0; i < 8; i++) c.ebest[kind][i] = e[i];
    }
    c.ecnt[kind] = has ? c.ecnt[kind] + 1u : 1u;
    return 1u << kind;
}
#if PG_MSX
// multi-seed exact pass: events carry one value per seed (scalar values broadcast)
__device__ __noinline__ u32 pg_event_ms(PgCold& c, u32 evm, u32 kind, u32 round, u32 arr, u32 addr, u32 ta,
                                        u32 tb, u32 site, const u32* va, u32 vb);
__device__ __forceinline__ u32 pg_event_msc(PgCold& c, u32 evm, u32 kind, u32 round, u32 arr, u32 addr, u32 ta,
                                            u32 tb, u32 site, u32 va, u32 vb) {
    u32 v[PG_MS];
    PG_S_LOOP v[_s] = va;
    return pg_event_ms(c, evm, kind, round, arr, addr, ta, tb, site, v, vb);
}
#define PG_EVENT(t, c, ...) ((t).evm |= pg_event_msc((c), (t).evm, __VA_ARGS__))
#elif PG_MS > 1
// multi-seed optimistic pass: an event flags the lane's instances, whose records the
// exact re-run then produces
#define PG_EVENT(t, c, ...) ((t).fl = 1u)
#else
#define PG_EVENT(t, c, ...) ((t).evm |= pg_event((c), (t).evm, __VA_ARGS__))
#endif

// stamps: step (20 bits, >= 1) and block-local tid (12 bits)
__device__ __forceinline__ u32 pg_stamp_min(const PgC& C, const PgT& t) { return C.smin | t.tlin; }
__device__ __forceinline__ u32 pg_stamp_max(const PgC& C, const PgT& t) { return C.smax | t.tlin; }
__device__ __forceinline__ u32 pg_owner_step(u32 own) { return 0xFFFFFu - (own >> 12); }

__device__ __forceinline__ u32* pg_sh(const PgT& t, u32 off) { return (u32*)(pg_dsmem + t.sg + off); }

// Optimistic pass, reader side of the RW check (one atomic per read): a cell of the round's
// parity set keeps the LAST reader's stamp (R, atomicExch; the rmin words) and a flag that
// a second, different reader of the same round came by (M = the round's smax tag; the rmax
// words).  After the barrier the writer w sees a race iff R is of this round and
// (R != w or M flagged): with two or more distinct readers some exchange returns another
// reader's stamp of the round and sets M; a single reader r != w leaves R = r.
__device__ __forceinline__ void pg_fread(u32* R, u32* M, u32 smax, u32 tlin) {
    const u32 me = smax | tlin;
    const u32 old = atomicExch(R, me);
    if (old != me && (old ^ me) < 0x1000u) *M = smax;
}

#ifndef PG_FAST
#define PG_FAST 0
#endif
#if PG_FAST
// Optimistic pass: stores commit in place and every round ends at one
// barrier.  That equals the round semantics X3/X4 whenever no race occurs, so the pass
// only has to DETECT that a race may have occurred; the instance is then re-run by the
// exact protocol.  A second writer of a cell in a round sees the first one's owner stamp
// in atomicMin's return value (WW).  Readers stamp the cell (reader stamps of the round's
// parity set, step & 1); after the round's barrier every writer re-reads the reader
// stamps of the cells it wrote - all reads of the round are visible then, whether they
// came before or after the write - while the next round stamps the other set (RW).
__shared__ u32 pg_sAbort;   // some thread of the CTA flagged (CTA-wide blocks)
#endif

// ------------------------------------------------------------------ bank / coalescing (X9, H6)
// wgt: instances this warp access stands for (multi-seed lanes: the group's seeds)
__device__ __forceinline__ void pg_site_stat(u64* st, u32 space, u32 bad, u32 metric, u32 ideal, u32 lanes, u32 wgt) {
    // [space, n_acc, n_bad, max, sum, sum_ideal, sum_lanes, 0]
    st[0] = space;
    atomicAdd(&st[1], (u64)wgt);
    if (bad) atomicAdd(&st[2], (u64)wgt);
    atomicMax(&st[3], (u64)metric);
    atomicAdd(&st[4], (u64)metric * wgt);
    atomicAdd(&st[5], (u64)ideal * wgt);
    atomicAdd(&st[6], (u64)lanes * wgt);
}
#if PG_MSX
#define PG_EVENT_RAW(c, evm, ...) pg_event_msc((c), (evm), __VA_ARGS__)
#else
#define PG_EVENT_RAW(c, evm, ...) pg_event((c), (evm), __VA_ARGS__)
#endif

// All 32 lanes of the warp call these together (the generated code keeps warps
// converged around every access site).
__device__ __noinline__ u32 pg_bank_shared(u32 round, u32 lane, u32 ekey0, u32 tlin, u32 gtid, PgCold& c, u32 evm,
                                           u64* sstats, u32 active, u32 rec, u32 flat, u32 site, u32 wgt = 1u) {
    u32 ekey = ekey0;
    if (PG_BANK16) ekey = ekey * 2u + ((tlin >> 4) & 1u);
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
    const u32 ta = __reduce_min_sync(seg, (active && flat == astar) ? gtid : PG_NEVER);
    const u32 tb = __reduce_min_sync(seg, (active && bank == bstar && flat != astar) ? gtid : PG_NEVER);
    if (amask && lane == (u32)(__ffs(amask) - 1)) {
        if (sstats && site < PG_NSTATS) pg_site_stat(sstats + site * 8, 1, deg > 1, deg, 1, __popc(amask), wgt);
        if (deg > 1) return PG_EVENT_RAW(c, evm, PGK_BANK, round, rec, astar, ta, tb, site, deg, 0);
    }
    return 0u;
}

__device__ __noinline__ u32 pg_coal_global(u32 round, u32 lane, u32 ekey, u32 gtid, PgCold& c, u32 evm,
                                           u64* sstats, u32 active, u32 rec, u32 flat, u32 site, u32 wgt = 1u) {
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
    const u32 ta = __reduce_min_sync(seg, active ? gtid : PG_NEVER);
    const u32 tb = __reduce_max_sync(seg, active ? gtid : 0u);
    if (amask && lane == (u32)(__ffs(amask) - 1)) {
        if (sstats && site < PG_NSTATS)
            pg_site_stat(sstats + site * 8, 2, sectors > ideal, sectors, ideal, __popc(amask), wgt);
        if (sectors > ideal) return PG_EVENT_RAW(c, evm, PGK_UNCOAL, round, rec, amin, ta, tb, site, sectors, ideal);
    }
    return 0u;
}

// ------------------------------------------------------------------ loads / stores
__device__ __forceinline__ u32 pg_log_find(const PgT& t, const PgCold& c, u32 cell, u32& v) {
    if (t.nlog == 0u) return 0u;
    if (t.l0cell == cell) {
        v = t.l0val;
        return 1u;
    }
    for (u32 i = 1; i < t.nlog; i++)
        if (c.lcell[i] == cell) {
            v = c.lval[i];
            return 1u;
        }
    return 0u;
}

// Returns the new log length, or PG_NEVER when the write-log limit dropped the write
// (X19; the caller records the LIMIT event).
__device__ __noinline__ u32 pg_log_write_slow(u32 nlog, PgCold& c, u32 cell, u32 val, u32 site) {
    for (u32 i = 1; i < nlog; i++) {
        if (c.lcell[i] == cell) {
            c.lval[i] = val;
            c.lsite[i] = (u16)site;
            return nlog;
        }
    }
    if (nlog >= PG_WMAX) return PG_NEVER;
    c.lcell[nlog] = cell;
    c.lval[nlog] = val;
    c.lsite[nlog] = (u16)site;
    return nlog + 1u;
}

// Returns 1 when the cell entered the log (its first store of the round: the claim).
__device__ __forceinline__ u32 pg_log_write(PgC& C, PgT& t, PgCold& c, u32 cell, u32 val, u32 site, u32 rec,
                                            u32 flat) {
    if (t.nlog == 0u) {
        t.l0cell = cell;
        t.l0val = val;
        t.l0site = site;
        t.nlog = 1u;
        return 1u;
    } else if (t.l0cell == cell) {
        t.l0val = val;
        t.l0site = site;
    } else {
        const u32 n = pg_log_write_slow(t.nlog, c, cell, val, site);
        if (n == PG_NEVER) PG_EVENT(t, c, PGK_LIMIT, C.round, rec, flat, t.gtid, PG_NEVER, site, 1, 0);
        else {
            const u32 fresh = n != t.nlog;
            t.nlog = n;
            return fresh;
        }
    }
    return 0u;
}

// Stamps of a global array the kernel writes: in the instance arena, or - single-block
// launches (PgArr flags bit 1, PgSA::gsh) - in the group's shared region, where they cost
// shared-memory atomics instead of L2 atomics (no other block can touch the cells)
#ifdef PG_S_T
#define PG_GSH(A) ((u32)PgSA<A>::gsh)
#else
#define PG_GSH(A) ((pg_sL.arr[A].flags >> 1) & 1u)
#endif
// Shared arrays whose stores are all at index tid.x in a one-dimensional block (PgArr flags
// bit 2, PgSA::tp; pg_ir_thread_private): no two threads store to one cell, so no WW race
// on them - stores take a plain owner stamp, no claim, and a check reads only reader stamps
#ifdef PG_S_T
#define PG_TP(A) ((u32)PgSA<A>::tp)
#define PG_TP_CONST(A) (PgSA<A>::tp != 0u)   // (a template argument: shape variants only)
#else
#define PG_TP(A) ((pg_sL.arr[A].flags >> 2) & 1u)
#define PG_TP_CONST(A) false
#endif
template <int A> __device__ __forceinline__ u32* pg_gown(const PgT& t) {
    return PG_GSH(A) ? pg_sh(t, PG_SH(A, s_own)) : t.arena + PG_ARR(A).off_own;
}
template <int A> __device__ __forceinline__ u32* pg_gwmax(const PgT& t) {
    return PG_GSH(A) ? pg_sh(t, PG_SH(A, s_wmax)) : t.arena + PG_ARR(A).off_wmax;
}
template <int A> __device__ __forceinline__ u32* pg_grmin(const PgT& t) {
    return PG_GSH(A) ? pg_sh(t, PG_SH(A, s_rmin)) : t.arena + PG_ARR(A).off_rmin;
}
template <int A> __device__ __forceinline__ u32* pg_grmax(const PgT& t) {
    return PG_GSH(A) ? pg_sh(t, PG_SH(A, s_rmax)) : t.arena + PG_ARR(A).off_rmax;
}

// Claim (exact protocol): atomicMin on the cell's claim stamp (newest round wins over stale
// stamps, the min tid wins within the round) plus atomicMax for WW detection.  Shared arrays
// claim into s_clm when claims happen at store time (PG_CAS: s_own keeps the committed owner
// that loads of the round consult), into s_own otherwise; global owner words are not read
// during a round outside the data-flow dump.
template <int A>
__device__ __forceinline__ void pg_claim_sh(const PgC& C, const PgT& t, u32 flat) {
    if (PG_TP(A)) return;   // (the writer owns the cell: the check commits it, no WW possible)
    atomicMin(pg_sh(t, PG_CAS ? PG_SH(A, s_clm) : PG_SH(A, s_own)) + flat, pg_stamp_min(C, t));
#if PG_RACECHK
    if (PG_T > 1u) atomicMax(pg_sh(t, PG_SH(A, s_wmax)) + flat, pg_stamp_max(C, t));
#endif
}
template <int A>
__device__ __forceinline__ void pg_claim_gt(const PgC& C, const PgT& t, u32 flat) {
    atomicMin(pg_gown<A>(t) + flat, pg_stamp_min(C, t));
#if PG_RACECHK
    if (PG_T > 1u) atomicMax(pg_gwmax<A>(t) + flat, pg_stamp_max(C, t));
#endif
}

#if PG_DATAFLOW
struct PgDf {
    u32* rows;
    u32* count;
    u64 seed_base;
    u32 cap;
};
__shared__ PgDf pg_sDf;  // data-flow recorder of this CTA
#define PG_HIST_R 64u   // rounds per block the VC-literal history keeps
#if PG_VCLIT
// GPU VC-literal mode: the
// writer of a read found by enumerating, for every earlier round (latest first; shared cells:
// this block's rounds, global cells: every block run so far, in bid order), every thread s
// of that round and testing "s wrote the cell" on s's logged writes of the round - the
// instantiated p(s) ∧ a = e(s) - instead of the owner stamps.  It must equal the data-flow
// row's owner-stamp writer (min s under WW); disagreements are counted (header word 1).
__device__ __noinline__ void pg_vclit(const PgC& C, const PgT& t, u32 cell, u32 glob, u32 src, u32 wb, u32 wr,
                                      u32 wg) {
    const u32 T = PG_T, HW = 1u + (u32)PG_WMAX;
    const u32* hist = t.arena + pg_sL.off_hist;
    const u32* hr = t.arena + pg_sL.off_hround;
    u32 fb = PG_NEVER, fr = PG_NEVER, fs = PG_NEVER;
    for (int b = (int)t.blk; b >= 0 && fs == PG_NEVER; b--) {
        if (!glob && (u32)b != t.blk) break;
        const u32 nr = (u32)b == t.blk ? C.round : hr[b];
        for (int r = (int)nr - 1; r >= 0 && fs == PG_NEVER; r--) {
            if ((u32)r >= PG_HIST_R) {   // (a round the history does not keep)
                atomicAdd(pg_sDf.count + 2, 1u);
                continue;
            }
            for (u32 s = 0; s < T; s++) {
                const u32* e = hist + (((u64)b * PG_HIST_R + (u32)r) * T + s) * HW;
                const u32 n = min(e[0], (u32)PG_WMAX);
                for (u32 i = 0; i < n; i++)
                    if (e[1 + i] == cell) {
                        fs = min(fs, s);
                        break;
                    }
            }
            if (fs != PG_NEVER) {
                fb = (u32)b;
                fr = (u32)r;
            }
        }
    }
    const bool ok = src == 0u ? fs == PG_NEVER : (fb == wb && fr == wr && fb * T + fs == wg);
    atomicAdd(pg_sDf.count + 3, 1u);
    if (!ok) atomicAdd(pg_sDf.count + 1, 1u);
}
#endif
__device__ __noinline__ void pg_df_row(const PgC& C, const PgT& t, u32 site, u32 rec, u32 flat, u32 src, u32 wb, u32 wr,
                                       u32 wg, u32 cell, u32 glob) {
#if PG_VCLIT
    if (src != 2u) pg_vclit(C, t, cell, glob, src, wb, wr, wg);
#endif
    const u32 i = atomicAdd(pg_sDf.count, 1u);
    if (i >= pg_sDf.cap) return;
    u32* r = pg_sDf.rows + (u64)i * 12u;
    r[0] = pg_sW.launch;
    r[1] = (u32)(t.seed - pg_sDf.seed_base);
    r[2] = t.blk; r[3] = C.round; r[4] = t.gtid; r[5] = site; r[6] = rec; r[7] = flat;
    r[8] = src; r[9] = wb; r[10] = wr; r[11] = wg;
}
// writer of a committed global cell: last committer (gtid) and the round of its stamp
__device__ __forceinline__ void pg_df_global(const PgC& C, const PgT& t, u32 site, u32 rec, u32 flat, u32 lw, u32 own,
                                             u64 off_step0, u32 cell) {
    if (!lw) { pg_df_row(C, t, site, rec, flat, 0u, PG_NEVER, PG_NEVER, PG_NEVER, cell, 1u); return; }
    const u32 wg = lw - 1u, wb = wg / PG_T;
    const u32 s0 = wb == t.blk ? C.step0 : t.arena[off_step0 + wb];
    pg_df_row(C, t, site, rec, flat, 1u, wb, pg_owner_step(own) - s0, wg, cell, 1u);
}
#endif

__device__ __forceinline__ u32 pg_poison_sh(const PgT& t, u32 rec, u32 flat) {
    return pg_m(pg_rand32(t.seed, 0x8000u + (rec - 0x100u), ((u64)t.blk << 20) + flat));
}

// Shared array A: value and owner-stamp words in the group's region.
// RD: reader stamps kept (race checks on, array read and written);
// LOG: a load of A may follow a store to A in the same round (own-write lookup).
#if PG_FAST
// cold path of a shared load: out of bounds or never written (X5/X6): poison value and
// the event (returned as value | event bits << 32)
__device__ __noinline__ u64 pg_ld_sh_cold(PgCold& c, u32 evm, u64 seed, u32 blk, u32 rec, u32 flat, u32 round,
                                         u32 gtid, u32 site, u32 oob) {
    const u32 pv = pg_m(pg_rand32(seed, 0x8000u + (rec - 0x100u), ((u64)blk << 20) + flat));
    u32 bits = 0u;
#if PG_OOBCHK
    bits = pg_event(c, evm, oob ? PGK_OOB : PGK_UNINIT, round, rec, flat, gtid, PG_NEVER, site, pv, 0);
#endif
    return (u64)pv | ((u64)bits << 32);
}
template <int A, bool RD, bool LOG>
__device__ __forceinline__ u32 pg_ld_sh(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site) {
    const u32 inb = flat < PG_SH(A, size);
#if PG_BANKCHK
    t.evm |= pg_bank_shared(C.round, t.lane, t.ekey, t.tlin, t.gtid, c, t.evm, ss, pe & inb, PG_ARR(A).rec_id, flat, site);
#endif
    u32 own = 0u, v = 0u;
    if (pe & inb) {
        if (RD && PG_T > 1u) {
            const u32 so = C.par * PG_SH(A, size) + flat;
            pg_fread(pg_sh(t, PG_SH(A, s_rmin)) + so, pg_sh(t, PG_SH(A, s_rmax)) + so, C.smax, t.tlin);
        }
        own = pg_sh(t, PG_SH(A, s_own))[flat];
        v = pg_sh(t, PG_SH(A, s_val))[flat];
    }
    if (pe & ((inb ^ 1u) | (u32)(own >= C.uthr))) {
        const u64 r = pg_ld_sh_cold(c, t.evm, t.seed, t.blk, PG_ARR(A).rec_id, flat, C.round, t.gtid, site, inb ^ 1u);
        t.evm |= (u32)(r >> 32);
        v = (u32)r;
    }
    return v;
}
#else
template <int A, bool RD, bool LOG>
__device__ __forceinline__ u32 pg_ld_sh(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site) {
    const u32 inb = flat < PG_SH(A, size);
#if PG_BANKCHK
    t.evm |= pg_bank_shared(C.round, t.lane, t.ekey, t.tlin, t.gtid, c, t.evm, ss, pe & inb, PG_ARR(A).rec_id, flat, site);
#endif
    if (!pe) return 0u;
    if (!inb) {
        const u32 pv = pg_poison_sh(t, PG_ARR(A).rec_id, flat);
#if PG_OOBCHK
        PG_EVENT(t, c, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, pv, 0);
#endif
        return pv;
    }
#if PG_RACECHK
    if (RD && PG_T > 1u) {
        atomicMin(pg_sh(t, PG_SH(A, s_rmin)) + flat, pg_stamp_min(C, t));
        atomicMax(pg_sh(t, PG_SH(A, s_rmax)) + flat, pg_stamp_max(C, t));
    }
#endif
    u32 v;
    if (LOG && pg_log_find(t, c, ((u32)A << 24) | flat, v)) {
#if PG_DATAFLOW
        pg_df_row(C, t, site, PG_ARR(A).rec_id, flat, 2u, t.blk, C.round, t.gtid, ((u32)A << 24) | flat, 0u);
#endif
        return v;
    }
    const u32 own = pg_sh(t, PG_SH(A, s_own))[flat];
    if (own >= C.uthr) {  // never written in this block (X6)
        const u32 pv = pg_poison_sh(t, PG_ARR(A).rec_id, flat);
#if PG_OOBCHK
        PG_EVENT(t, c, PGK_UNINIT, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, pv, 0);
#endif
#if PG_DATAFLOW
        pg_df_row(C, t, site, PG_ARR(A).rec_id, flat, 0u, PG_NEVER, PG_NEVER, PG_NEVER, ((u32)A << 24) | flat, 0u);
#endif
        return pv;
    }
#if PG_DATAFLOW
    pg_df_row(C, t, site, PG_ARR(A).rec_id, flat, 1u, t.blk, pg_owner_step(own) - C.step0,
              t.blk * PG_T + (own & 0xFFFu), ((u32)A << 24) | flat, 0u);
#endif
    return pg_sh(t, PG_SH(A, s_val))[flat];
}
#endif

#if PG_FAST
// write log of the optimistic pass: cells whose readers are checked after the barrier
// (low 16 bits: logged cells; high 16 bits: stores this round, X19's W_max)
__device__ __forceinline__ void pg_flog(PgT& t, PgCold& c, u32 cell) {
    const u32 n = t.nlog & 0xFFFFu;
    if (n == 0u) {
        t.l0cell = cell;
        t.nlog += 1u;
    } else if (t.l0cell != cell) {
        const u32 m = pg_log_write_slow(n, c, cell, 0u, 0u);
        if (m == PG_NEVER) t.fl = 1u;
        else t.nlog += m - n;
    }
}
__device__ __forceinline__ void pg_fcount(PgT& t) {
    t.nlog += 0x10000u;
    t.fl |= (t.nlog >> 16) > (u32)PG_WMAX;   // more stores than the write log holds: LIMIT is decided exactly
}
// in-place commit (optimistic pass): owner stamp (WW detection), value, reader check log
template <int A, bool RDA>
__device__ __forceinline__ void pg_commit_sh(const PgC& C, PgT& t, PgCold& c, u32 flat, u32 val) {
    u32* own = pg_sh(t, PG_SH(A, s_own)) + flat;
    const u32 me = C.smin | t.tlin;
    if (PG_T > 1u && !PG_TP(A)) {
        const u32 old = atomicMin(own, me);
        t.fl |= (old ^ me) - 1u < 0xFFFu;   // another writer's stamp of this round (WW)
    } else {
        *own = me;   // (one thread per block writes the cell: no claim)
    }
    if (PG_T > 1u && RDA) pg_flog(t, c, ((u32)A << 24) | flat);
    pg_sh(t, PG_SH(A, s_val))[flat] = val;
    pg_fcount(t);
}
// after the round's barrier: a reader of the round other than this thread (pg_fread: the
// last reader word R is of this round and another thread's, or a second reader was flagged)
__device__ __forceinline__ u32 pg_fast_rw(const PgC& C, const PgT& t, u32 R, u32 M) {
    const u32 a = R ^ (C.smax | t.tlin);
    return (a < 0x1000u) & ((a != 0u) | (M == C.smax));
}
template <int A>
__device__ __forceinline__ void pg_fcheck_sh(const PgC& C, PgT& t, u32 flat) {
    const u32 so = C.par * PG_SH(A, size) + flat;
    t.fl |= pg_fast_rw(C, t, pg_sh(t, PG_SH(A, s_rmin))[so], pg_sh(t, PG_SH(A, s_rmax))[so]);
}
template <int A>
__device__ __forceinline__ void pg_fcheck_gt(const PgC& C, PgT& t, u32 flat) {
    const u64 so = (u64)C.par * PG_ARR(A).size + flat;
    t.fl |= pg_fast_rw(C, t, pg_grmin<A>(t)[so], pg_grmax<A>(t)[so]);
}
// (C still describes the round just finished)
template <class K>
__device__ __forceinline__ void pg_fcheck_all(const PgC& C, PgT& t, PgCold& c) {
    const u32 n = t.nlog & 0xFFFFu;
    if (n == 0u) return;
    K::fcheck_one(C, t, t.l0cell);
    for (u32 i = 1; i < n; i++) K::fcheck_one(C, t, c.lcell[i]);
}
#endif

template <int A, bool RDA = false>
__device__ __forceinline__ void pg_st_sh(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 val, u32 site) {
    const u32 inb = flat < PG_SH(A, size);
#if PG_BANKCHK
    t.evm |= pg_bank_shared(C.round, t.lane, t.ekey, t.tlin, t.gtid, c, t.evm, ss, pe & inb, PG_ARR(A).rec_id, flat, site);
#endif
    if (!pe) return;
    if (!inb) {
#if PG_OOBCHK
        PG_EVENT(t, c, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, val, 1);
#endif
        return;
    }
#if PG_FAST
    pg_commit_sh<A, RDA>(C, t, c, flat, val);
#else
    if (pg_log_write(C, t, c, ((u32)A << 24) | flat, val, site, PG_ARR(A).rec_id, flat) && PG_CAS && PG_T > 1u)
        pg_claim_sh<A>(C, t, flat);
#endif
}

#if PG_MS > 1
// ------------------------------------------------------------------ multi-seed lanes
// Optimistic pass of a seed-oblivious kernel (codegen seed_oblivious): the PG_MS seeds of
// a group take the same accesses, so one lane evaluates the address, guard, stamp and
// race logic once and carries PG_MS values.  Shared values are laid out [cell][seed]
// (one 128-bit access for PG_MS = 4); stamps are per cell as before.  Anything that
// would be an event (OOB, UNINIT, LIMIT, a race) flags the group's instances, which the
// exact single-seed re-run then evaluates and records.
__device__ __forceinline__ void pg_vld(const u32* p, u32 (&v)[PG_MS]) {
#if PG_MS == 16
#pragma unroll
    for (int h = 0; h < 4; h++) {
        const uint4 q = *(const uint4*)(p + 4 * h);
        v[4 * h] = q.x; v[4 * h + 1] = q.y; v[4 * h + 2] = q.z; v[4 * h + 3] = q.w;
    }
#elif PG_MS == 8
    const uint4 q = *(const uint4*)p, r = *(const uint4*)(p + 4);
    v[0] = q.x; v[1] = q.y; v[2] = q.z; v[3] = q.w; v[4] = r.x; v[5] = r.y; v[6] = r.z; v[7] = r.w;
#elif PG_MS == 4
    const uint4 q = *(const uint4*)p;
    v[0] = q.x; v[1] = q.y; v[2] = q.z; v[3] = q.w;
#elif PG_MS == 2
    const uint2 q = *(const uint2*)p;
    v[0] = q.x; v[1] = q.y;
#else
    PG_S_LOOP v[_s] = p[_s];
#endif
}
__device__ __forceinline__ void pg_vst(u32* p, const u32 (&v)[PG_MS]) {
#if PG_MS == 16
#pragma unroll
    for (int h = 0; h < 4; h++) *(uint4*)(p + 4 * h) = make_uint4(v[4 * h], v[4 * h + 1], v[4 * h + 2], v[4 * h + 3]);
#elif PG_MS == 8
    *(uint4*)p = make_uint4(v[0], v[1], v[2], v[3]);
    *(uint4*)(p + 4) = make_uint4(v[4], v[5], v[6], v[7]);
#elif PG_MS == 4
    *(uint4*)p = make_uint4(v[0], v[1], v[2], v[3]);
#elif PG_MS == 2
    *(uint2*)p = make_uint2(v[0], v[1]);
#else
    PG_S_LOOP p[_s] = v[_s];
#endif
}
#if PG_FAST
template <int A, bool RD, bool LOG>
__device__ __forceinline__ void pg_ld_sh_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site,
                                            u32 (&v)[PG_MS]) {
    const u32 inb = flat < PG_SH(A, size);
    u32 own = 0u;
    if (pe & inb) {
        if (RD && PG_T > 1u) {
            const u32 so = C.par * PG_SH(A, size) + flat;
            pg_fread(pg_sh(t, PG_SH(A, s_rmin)) + so, pg_sh(t, PG_SH(A, s_rmax)) + so, C.smax, t.tlin);
        }
        own = pg_sh(t, PG_SH(A, s_own))[flat];
        pg_vld(pg_sh(t, PG_SH(A, s_val)) + flat * PG_MS, v);
    } else {
        PG_S_LOOP v[_s] = 0u;
    }
    t.fl |= pe & ((inb ^ 1u) | (u32)(own >= C.uthr));   // OOB / never written (X5, X6)
}
template <int A, bool RDA = false>
__device__ __forceinline__ void pg_st_sh_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat,
                                            const u32 (&val)[PG_MS], u32 site) {
    if (!pe) return;
    if (flat >= PG_SH(A, size)) {
        t.fl = 1u;
        return;
    }
    u32* own = pg_sh(t, PG_SH(A, s_own)) + flat;
    const u32 me = C.smin | t.tlin;
    if (PG_T > 1u && !PG_TP(A)) {
        const u32 old = atomicMin(own, me);
        t.fl |= (old ^ me) - 1u < 0xFFFu;   // another writer's stamp of this round (WW)
    } else {
        *own = me;   // (one thread per block writes the cell: no claim)
    }
    if (PG_T > 1u && RDA) pg_flog(t, c, ((u32)A << 24) | flat);
    pg_vst(pg_sh(t, PG_SH(A, s_val)) + flat * PG_MS, val);
    pg_fcount(t);
}
// global arrays: per-seed arenas for values and last writers (read per instance by K2b/K3);
// owner, reader and XB block stamps agree across the seeds and live in the group's first
// arena only (K1 initialises them there only, K2b flags the whole group)
template <int A>
__device__ __forceinline__ void pg_xb_mark_ms(const PgT& t, u32 flat) {
    if (pg_sL.nblocks > 1u && PG_ARR(A).off_xf != ~0ull) {   // (the group's first arena: every seed touches the same cells; K2b
                                //  decides for the whole group)
        atomicMin(t.arena + PG_ARR(A).off_xf + flat, t.blk + 1u);
        atomicMax(t.arena + PG_ARR(A).off_xl + flat, t.blk + 1u);
    }
}
template <int A, bool RD, bool LOG>
__device__ __forceinline__ void pg_ld_gt_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site,
                                            u32 (&v)[PG_MS]) {
    PG_S_LOOP v[_s] = 0u;
    if (!pe) return;
    if (flat >= PG_ARR(A).size) {
        t.fl = 1u;
        return;
    }
    pg_xb_mark_ms<A>(t, flat);
    if (RD && PG_T > 1u) {
        const u64 so = (u64)C.par * PG_ARR(A).size + flat;
        pg_fread(pg_grmin<A>(t) + so, pg_grmax<A>(t) + so, C.smax, t.tlin);
    }
    const u64 st = pg_sL.arena_stride;
    PG_S_LOOP if (_s < t.nsv) v[_s] = t.arena[_s * st + PG_ARR(A).off_val + flat];
}
template <int A, bool RDA = false>
__device__ __forceinline__ void pg_st_gt_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat,
                                            const u32 (&val)[PG_MS], u32 site) {
    if (!pe) return;
    if (flat >= PG_ARR(A).size) {
        t.fl = 1u;
        return;
    }
    pg_xb_mark_ms<A>(t, flat);
    u32* own = pg_gown<A>(t) + flat;
    const u32 me = C.smin | t.tlin;
    if (PG_T > 1u) {
        const u32 old = atomicMin(own, me);
        t.fl |= (old ^ me) - 1u < 0xFFFu;
        if (RDA) pg_flog(t, c, ((u32)A << 24) | flat);
    } else {
        *own = me;
    }
    const u64 st = pg_sL.arena_stride;
    PG_S_LOOP if (_s < t.nsv) t.arena[_s * st + PG_ARR(A).off_val + flat] = val[_s];
    // the last writer is the same in every seed of the group (same accesses): the group's first
    // arena keeps it (K2b and K3 read it there)
    t.arena[PG_ARR(A).off_lw + flat] = t.gtid + 1u;
    pg_fcount(t);
}
template <int A>
__device__ __forceinline__ void pg_ld_gi_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site,
                                            u32 (&v)[PG_MS]) {
    PG_S_LOOP v[_s] = 0u;
    if (!pe) return;
    if (flat >= PG_ARR(A).size) {
        t.fl = 1u;
        return;
    }
    const u32* p = t.input + PG_ARR(A).off_in + flat;
    const u64 st = pg_sL.input_stride;
    PG_S_LOOP v[_s] = __ldg(p + (u64)min(_s, t.nsv - 1u) * st);
}
#else   // PG_MSX: the exact protocol, PG_MS seeds per lane
// Per seed: write-log values, committed values, poison values and the events' value
// fields; once per cell: claims, owner / race stamps and the race decision.
__device__ __forceinline__ u64 pg_seed_of(const PgT& t, u32 s) { return t.seed + (u64)s * pg_sW.seed_jstep; }
__device__ __noinline__ u32 pg_event_ms(PgCold& c, u32 evm, u32 kind, u32 round, u32 arr, u32 addr, u32 ta,
                                        u32 tb, u32 site, const u32* va, u32 vb) {
    const u32 e[6] = {round, arr, addr, ta, tb, site};
    const u32 has = (evm >> kind) & 1u;
    const u64 pk = pg_pack(e);
    int cmp = -1;
    if (has) {
        const u64 bp = c.epk[kind];
        cmp = pk < bp ? -1 : pk > bp ? 1 : 0;   // (pg_pack is monotone: unequal packs decide)
        for (int i = 0; i < 6 && cmp == 0; i++)
            if (e[i] != c.ebest[kind][i]) cmp = e[i] < c.ebest[kind][i] ? -1 : 1;
    }
    const u32 nvx = evm ? c.vbx : 0u;   // (the thread's first event initialises vbx)
    if (cmp < 0) {
        c.epk[kind] = pk;
        for (int i = 0; i < 6; i++) c.ebest[kind][i] = e[i];
        PG_S_LOOP c.ebv[kind][_s] = va[_s];
        c.ebvb[kind] = vb;
        c.vbx = nvx & ~(1u << kind);
    } else if (cmp == 0) {   // same access: the per-seed values decide (X16 lexicographic order)
        if (!((nvx >> kind) & 1u) && vb == c.ebvb[kind]) {
            PG_S_LOOP if (va[_s] < c.ebv[kind][_s]) c.ebv[kind][_s] = va[_s];
        } else {   // (rare: val_b may now differ between seeds)
            if (!((nvx >> kind) & 1u)) PG_S_LOOP c.ebvs[kind][_s] = c.ebvb[kind];
            c.vbx = nvx | (1u << kind);
            PG_S_LOOP {
                if (va[_s] < c.ebv[kind][_s] || (va[_s] == c.ebv[kind][_s] && vb < c.ebvs[kind][_s])) {
                    c.ebv[kind][_s] = va[_s];
                    c.ebvs[kind][_s] = vb;
                }
            }
        }
    }
    c.ecnt[kind] = has ? c.ecnt[kind] + 1u : 1u;
    return 1u << kind;
}
__device__ __forceinline__ u32 pg_log_find_ms(const PgT& t, const PgCold& c, u32 cell, u32 (&v)[PG_MS]) {
    if (t.nlog == 0u) return 0u;
    if (t.l0cell == cell) {
        PG_S_LOOP v[_s] = t.l0v[_s];
        return 1u;
    }
    for (u32 i = 1; i < t.nlog; i++)
        if (c.lcell[i] == cell) {
            PG_S_LOOP v[_s] = c.lvs[i][_s];
            return 1u;
        }
    return 0u;
}
__device__ __noinline__ u32 pg_log_write_slow_ms(u32 nlog, PgCold& c, u32 cell, const u32* val, u32 site) {
    for (u32 i = 1; i < nlog; i++) {
        if (c.lcell[i] == cell) {
            PG_S_LOOP c.lvs[i][_s] = val[_s];
            c.lsite[i] = (u16)site;
            return nlog;
        }
    }
    if (nlog >= PG_WMAX) return PG_NEVER;
    c.lcell[nlog] = cell;
    PG_S_LOOP c.lvs[nlog][_s] = val[_s];
    c.lsite[nlog] = (u16)site;
    return nlog + 1u;
}
__device__ __forceinline__ u32 pg_log_write_ms(PgC& C, PgT& t, PgCold& c, u32 cell, const u32 (&val)[PG_MS],
                                               u32 site, u32 rec, u32 flat) {
    if (t.nlog == 0u) {
        t.l0cell = cell;
        PG_S_LOOP t.l0v[_s] = val[_s];
        t.l0site = site;
        t.nlog = 1u;
        return 1u;
    } else if (t.l0cell == cell) {
        PG_S_LOOP t.l0v[_s] = val[_s];
        t.l0site = site;
    } else {
        const u32 n = pg_log_write_slow_ms(t.nlog, c, cell, val, site);
        if (n == PG_NEVER) PG_EVENT(t, c, PGK_LIMIT, C.round, rec, flat, t.gtid, PG_NEVER, site, 1, 0);
        else {
            const u32 fresh = n != t.nlog;
            t.nlog = n;
            return fresh;
        }
    }
    return 0u;
}
template <int A, bool RD, bool LOG>
__device__ __forceinline__ void pg_ld_sh_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site,
                                            u32 (&v)[PG_MS]) {
#if PG_BANKCHK
    t.evm |= pg_bank_shared(C.round, t.lane, t.ekey, t.tlin, t.gtid, c, t.evm, ss, pe & (flat < PG_SH(A, size)),
                            PG_ARR(A).rec_id, flat, site, t.nsv);
#endif
    PG_S_LOOP v[_s] = 0u;
    if (!pe) return;
    const u32 rec = PG_ARR(A).rec_id;
    if (flat >= PG_SH(A, size)) {
        PG_S_LOOP v[_s] = pg_m(pg_rand32(pg_seed_of(t, _s), 0x8000u + (rec - 0x100u), ((u64)t.blk << 20) + flat));
#if PG_OOBCHK
        t.evm |= pg_event_ms(c, t.evm, PGK_OOB, C.round, rec, flat, t.gtid, PG_NEVER, site, v, 0);
#endif
        return;
    }
#if PG_RACECHK
    if (RD && PG_T > 1u) {
        atomicMin(pg_sh(t, PG_SH(A, s_rmin)) + flat, pg_stamp_min(C, t));
        atomicMax(pg_sh(t, PG_SH(A, s_rmax)) + flat, pg_stamp_max(C, t));
    }
#endif
    if (LOG && pg_log_find_ms(t, c, ((u32)A << 24) | flat, v)) return;
    const u32 own = pg_sh(t, PG_SH(A, s_own))[flat];
    if (own >= C.uthr) {  // never written in this block (X6)
        PG_S_LOOP v[_s] = pg_m(pg_rand32(pg_seed_of(t, _s), 0x8000u + (rec - 0x100u), ((u64)t.blk << 20) + flat));
#if PG_OOBCHK
        t.evm |= pg_event_ms(c, t.evm, PGK_UNINIT, C.round, rec, flat, t.gtid, PG_NEVER, site, v, 0);
#endif
        return;
    }
    pg_vld(pg_sh(t, PG_SH(A, s_val)) + flat * PG_MS, v);
}
template <int A, bool RDA = false>
__device__ __forceinline__ void pg_st_sh_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat,
                                            const u32 (&val)[PG_MS], u32 site) {
#if PG_BANKCHK
    t.evm |= pg_bank_shared(C.round, t.lane, t.ekey, t.tlin, t.gtid, c, t.evm, ss, pe & (flat < PG_SH(A, size)),
                            PG_ARR(A).rec_id, flat, site, t.nsv);
#endif
    if (!pe) return;
    if (flat >= PG_SH(A, size)) {
#if PG_OOBCHK
        t.evm |= pg_event_ms(c, t.evm, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, val, 1);
#endif
        return;
    }
    if (pg_log_write_ms(C, t, c, ((u32)A << 24) | flat, val, site, PG_ARR(A).rec_id, flat) && PG_CAS && PG_T > 1u)
        pg_claim_sh<A>(C, t, flat);
}
template <int A>
__device__ __forceinline__ void pg_xb_mark_ms(const PgT& t, u32 flat) {
    if (pg_sL.nblocks > 1u && PG_ARR(A).off_xf != ~0ull) {   // (the group's first arena: every seed touches the same cells; K2b
                                //  decides for the whole group)
        atomicMin(t.arena + PG_ARR(A).off_xf + flat, t.blk + 1u);
        atomicMax(t.arena + PG_ARR(A).off_xl + flat, t.blk + 1u);
    }
}
template <int A, bool RD, bool LOG>
__device__ __forceinline__ void pg_ld_gt_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site,
                                            u32 (&v)[PG_MS]) {
#if PG_COALCHK
    t.evm |= pg_coal_global(C.round, t.lane, t.ekey, t.gtid, c, t.evm, ss, pe & (flat < PG_ARR(A).size),
                            PG_ARR(A).rec_id, flat, site, t.nsv);
#endif
    PG_S_LOOP v[_s] = 0u;
    if (!pe) return;
    if (flat >= PG_ARR(A).size) {
        PG_S_LOOP v[_s] = pg_m(pg_rand32(pg_seed_of(t, _s), PG_ARR(A).gid, flat));
#if PG_OOBCHK
        t.evm |= pg_event_ms(c, t.evm, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, v, 0);
#endif
        return;
    }
    pg_xb_mark_ms<A>(t, flat);
#if PG_RACECHK
    if (RD && PG_T > 1u) {
        atomicMin(pg_grmin<A>(t) + flat, pg_stamp_min(C, t));
        atomicMax(pg_grmax<A>(t) + flat, pg_stamp_max(C, t));
    }
#endif
    if (LOG && pg_log_find_ms(t, c, ((u32)A << 24) | flat, v)) return;
    const u64 st = pg_sL.arena_stride;
    PG_S_LOOP if (_s < t.nsv) v[_s] = t.arena[_s * st + PG_ARR(A).off_val + flat];
}
template <int A, bool RDA = false>
__device__ __forceinline__ void pg_st_gt_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat,
                                            const u32 (&val)[PG_MS], u32 site) {
#if PG_COALCHK
    t.evm |= pg_coal_global(C.round, t.lane, t.ekey, t.gtid, c, t.evm, ss, pe & (flat < PG_ARR(A).size),
                            PG_ARR(A).rec_id, flat, site, t.nsv);
#endif
    if (!pe) return;
    if (flat >= PG_ARR(A).size) {
#if PG_OOBCHK
        t.evm |= pg_event_ms(c, t.evm, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, val, 1);
#endif
        return;
    }
    pg_xb_mark_ms<A>(t, flat);
    if (pg_log_write_ms(C, t, c, ((u32)A << 24) | flat, val, site, PG_ARR(A).rec_id, flat) && PG_CAS && PG_T > 1u)
        pg_claim_gt<A>(C, t, flat);
}
template <int A>
__device__ __forceinline__ void pg_ld_gi_ms(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site,
                                            u32 (&v)[PG_MS]) {
#if PG_COALCHK
    t.evm |= pg_coal_global(C.round, t.lane, t.ekey, t.gtid, c, t.evm, ss, pe & (flat < PG_ARR(A).size),
                            PG_ARR(A).rec_id, flat, site, t.nsv);
#endif
    PG_S_LOOP v[_s] = 0u;
    if (!pe) return;
    if (flat >= PG_ARR(A).size) {
        PG_S_LOOP v[_s] = pg_m(pg_rand32(pg_seed_of(t, _s), PG_ARR(A).gid, flat));
#if PG_OOBCHK
        t.evm |= pg_event_ms(c, t.evm, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, v, 0);
#endif
        return;
    }
    const u32* p = t.input + PG_ARR(A).off_in + flat;
    const u64 st = pg_sL.input_stride;
    PG_S_LOOP v[_s] = __ldg(p + (u64)min(_s, t.nsv - 1u) * st);
}
// round end of the exact protocol: the owner commits every seed's value; race decisions
// are per cell, their records carry each seed's value
__device__ PG_RC_INLINE u32 pg_race_check_ms(u32 round, u32 step, u32 tlin, u32 gtid, PgCold& c, u32 evm,
                                             const u32* val, u32 site, u32 rec, u32 flat, u32 own, u32 wmax,
                                             u32 has_readers, u32 rmin, u32 rmax) {
    const u32 base = gtid - tlin;
    const u32 w0 = own & 0xFFFu, w1 = wmax & 0xFFFu;
    if (w1 != w0 && tlin == w0) evm |= pg_event_ms(c, evm, PGK_WW, round, rec, flat, gtid, base + w1, site, val, 0);
    if (has_readers && (rmax >> 12) == step) {
        const u32 r0 = rmin & 0xFFFu, r1 = rmax & 0xFFFu;
        if (!(r0 == r1 && w0 == w1 && r0 == w0)) {
            u32 ta, tb;
            if (r0 != w0) { ta = w0; tb = r0; }
            else if (r1 != w0) { ta = w0; tb = r1; }
            else { ta = w1; tb = r0; }
            if (tlin == ta) evm |= pg_event_ms(c, evm, PGK_RW, round, rec, flat, base + ta, base + tb, site, val, 0);
        }
    }
    return evm;
}
template <int A, bool RD>
__device__ __forceinline__ void pg_check_sh_ms(const PgC& C, PgT& t, PgCold& c, u32 flat, const u32* val, u32 site) {
    u32 v[PG_MS];
    PG_S_LOOP v[_s] = val[_s];
    if (PG_T == 1u) {
        pg_sh(t, PG_SH(A, s_own))[flat] = pg_stamp_min(C, t);
        pg_vst(pg_sh(t, PG_SH(A, s_val)) + flat * PG_MS, v);
        return;
    }
    // (thread-private stores: the writer owns its cell, no claim was made)
    const u32 own = PG_TP(A) ? pg_stamp_min(C, t) : pg_sh(t, PG_CAS ? PG_SH(A, s_clm) : PG_SH(A, s_own))[flat];
    if (own == pg_stamp_min(C, t)) {
        pg_vst(pg_sh(t, PG_SH(A, s_val)) + flat * PG_MS, v);
        if (PG_CAS || PG_TP(A)) pg_sh(t, PG_SH(A, s_own))[flat] = own;
    }
#if PG_RACECHK
    if (PG_T > 1u) {
        const u32 wmax = PG_TP(A) ? pg_stamp_max(C, t) : pg_sh(t, PG_SH(A, s_wmax))[flat];
        const u32 rmin = RD ? pg_sh(t, PG_SH(A, s_rmin))[flat] : 0u;
        const u32 rmax = RD ? pg_sh(t, PG_SH(A, s_rmax))[flat] : 0u;
        if ((wmax & 0xFFFu) != (own & 0xFFFu) ||
            (RD && (rmax >> 12) == C.step && (((rmin ^ own) | (rmax ^ own)) & 0xFFFu)))
            t.evm = pg_race_check_ms(C.round, C.step, t.tlin, t.gtid, c, t.evm, val, site, PG_ARR(A).rec_id, flat,
                                     own, wmax, RD, rmin, rmax);
    }
#endif
}
template <int A, bool RD>
__device__ __forceinline__ void pg_check_gt_ms(const PgC& C, PgT& t, PgCold& c, u32 flat, const u32* val, u32 site) {
    const u64 st = pg_sL.arena_stride;
    if (PG_T == 1u) {
        pg_gown<A>(t)[flat] = pg_stamp_min(C, t);
        PG_S_LOOP {
            if (_s < t.nsv) {
                t.arena[_s * st + PG_ARR(A).off_val + flat] = val[_s];
                t.arena[_s * st + PG_ARR(A).off_lw + flat] = t.gtid + 1u;
            }
        }
        return;
    }
    const u32 own = pg_gown<A>(t)[flat];
    if (own == pg_stamp_min(C, t)) {
        PG_S_LOOP {
            if (_s < t.nsv) {
                t.arena[_s * st + PG_ARR(A).off_val + flat] = val[_s];
                t.arena[_s * st + PG_ARR(A).off_lw + flat] = t.gtid + 1u;
            }
        }
    }
#if PG_RACECHK
    if (PG_T > 1u) {
        const u32 wmax = pg_gwmax<A>(t)[flat];
        const u32 rmin = RD ? pg_grmin<A>(t)[flat] : 0u;
        const u32 rmax = RD ? pg_grmax<A>(t)[flat] : 0u;
        if ((wmax & 0xFFFu) != (own & 0xFFFu) ||
            (RD && (rmax >> 12) == C.step && (((rmin ^ own) | (rmax ^ own)) & 0xFFFu)))
            t.evm = pg_race_check_ms(C.round, C.step, t.tlin, t.gtid, c, t.evm, val, site, PG_ARR(A).rec_id, flat,
                                     own, wmax, RD, rmin, rmax);
    }
#endif
}
#endif   // PG_FAST
#endif

// XB bookkeeping (X4): first and last block that accessed a global cell.  Kept
// whenever the launch has more than one block (it also decides whether the
// block-parallel pass must be redone sequentially).
template <int A>
__device__ __forceinline__ void pg_xb_mark(const PgT& t, u32 flat) {
    if (pg_sL.nblocks > 1u && PG_ARR(A).off_xf != ~0ull) {   // (~0: block-private outputs, no XB)
        atomicMin(t.arena + PG_ARR(A).off_xf + flat, t.blk + 1u);
        atomicMax(t.arena + PG_ARR(A).off_xl + flat, t.blk + 1u);
    }
}

// Global array written by this kernel: values + owner stamps in the instance arena.
template <int A, bool RD, bool LOG>
__device__ __forceinline__ u32 pg_ld_gt(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site) {
    const u32 inb = flat < PG_ARR(A).size;
#if PG_COALCHK
    t.evm |= pg_coal_global(C.round, t.lane, t.ekey, t.gtid, c, t.evm, ss, pe & inb, PG_ARR(A).rec_id, flat, site);
#endif
    if (!pe) return 0u;
    if (!inb) {
        const u32 pv = pg_m(pg_rand32(t.seed, PG_ARR(A).gid, flat));
#if PG_OOBCHK
        PG_EVENT(t, c, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, pv, 0);
#endif
        return pv;
    }
    pg_xb_mark<A>(t, flat);
#if PG_FAST
    if (RD && PG_T > 1u) {
        const u64 so = (u64)C.par * PG_ARR(A).size + flat;
        pg_fread(pg_grmin<A>(t) + so, pg_grmax<A>(t) + so, C.smax, t.tlin);
    }
    return t.arena[PG_ARR(A).off_val + flat];
#else
#if PG_RACECHK
    if (RD && PG_T > 1u) {
        atomicMin(pg_grmin<A>(t) + flat, pg_stamp_min(C, t));
        atomicMax(pg_grmax<A>(t) + flat, pg_stamp_max(C, t));
    }
#endif
    u32 v;
    if (LOG && pg_log_find(t, c, ((u32)A << 24) | flat, v)) {
#if PG_DATAFLOW
        pg_df_row(C, t, site, PG_ARR(A).rec_id, flat, 2u, t.blk, C.round, t.gtid, ((u32)A << 24) | flat, 1u);
#endif
        return v;
    }
#if PG_DATAFLOW
    pg_df_global(C, t, site, PG_ARR(A).rec_id, flat, t.arena[PG_ARR(A).off_lw + flat],
                 t.arena[PG_ARR(A).off_own + flat], pg_sL.off_step0, ((u32)A << 24) | flat);
#endif
    return t.arena[PG_ARR(A).off_val + flat];
#endif
}

template <int A, bool RDA = false>
__device__ __forceinline__ void pg_st_gt(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 val, u32 site) {
    const u32 inb = flat < PG_ARR(A).size;
#if PG_COALCHK
    t.evm |= pg_coal_global(C.round, t.lane, t.ekey, t.gtid, c, t.evm, ss, pe & inb, PG_ARR(A).rec_id, flat, site);
#endif
    if (!pe) return;
    if (!inb) {
#if PG_OOBCHK
        PG_EVENT(t, c, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, val, 1);
#endif
        return;
    }
    pg_xb_mark<A>(t, flat);
#if PG_FAST
    {
        u32* own = pg_gown<A>(t) + flat;
        const u32 me = C.smin | t.tlin;
        if (PG_T > 1u) {
            const u32 old = atomicMin(own, me);
            t.fl |= (old ^ me) - 1u < 0xFFFu;
            if (RDA) pg_flog(t, c, ((u32)A << 24) | flat);
        } else {
            *own = me;
        }
        t.arena[PG_ARR(A).off_val + flat] = val;
        t.arena[PG_ARR(A).off_lw + flat] = t.gtid + 1u;
        pg_fcount(t);
    }
#else
    if (pg_log_write(C, t, c, ((u32)A << 24) | flat, val, site, PG_ARR(A).rec_id, flat) && PG_CAS && PG_T > 1u)
        pg_claim_gt<A>(C, t, flat);
#endif
}

// Global array this kernel only reads: the instance's input region.
template <int A>
__device__ __forceinline__ u32 pg_ld_gi(PgC& C, PgT& t, PgCold& c, u64* ss, u32 pe, u32 flat, u32 site) {
    const u32 inb = flat < PG_ARR(A).size;
#if PG_COALCHK
    t.evm |= pg_coal_global(C.round, t.lane, t.ekey, t.gtid, c, t.evm, ss, pe & inb, PG_ARR(A).rec_id, flat, site);
#endif
    if (!pe) return 0u;
    if (!inb) {
        const u32 pv = pg_m(pg_rand32(t.seed, PG_ARR(A).gid, flat));
#if PG_OOBCHK
        PG_EVENT(t, c, PGK_OOB, C.round, PG_ARR(A).rec_id, flat, t.gtid, PG_NEVER, site, pv, 0);
#endif
        return pv;
    }
#if PG_DATAFLOW
    pg_df_row(C, t, site, PG_ARR(A).rec_id, flat, 0u, PG_NEVER, PG_NEVER, PG_NEVER, ((u32)A << 24) | flat, 1u);
#endif
    return __ldg(t.input + PG_ARR(A).off_in + flat);
}

// Private (per-thread) array: bounds check only (X5); no races, no logging.
__device__ __forceinline__ u32 pg_priv_ok(PgC& C, PgT& t, PgCold& c, u32 pe, u32 flat, u32 size, u32 rec, u32 site,
                                          u32 val, u32 is_store) {
    if (!pe) return 0u;
    if (flat < size) return 1u;
#if PG_OOBCHK
    PG_EVENT(t, c, PGK_OOB, C.round, rec, flat, t.gtid, PG_NEVER, site, is_store ? val : 0u, is_store);
#endif
    return 0u;
}

// ------------------------------------------------------------------ loops (fuel, X19)
__device__ __forceinline__ void pg_tick(PgC& C, PgT& t, PgCold& c, u32 act) {
    if (act && ++t.fuel > C.fuel) {
        PG_EVENT(t, c, PGK_LIMIT, C.round, PG_NEVER, 0, t.gtid, PG_NEVER, PG_NEVER, 2, 0);
        t.live = 0;
    }
}

// ------------------------------------------------------------------ round end (H4)
// Claim: atomicMin on the owner stamp (newest round wins over stale stamps, the
// min tid wins within the round).  Check (after a barrier): the owner commits
// its value (and, for global arrays, itself as last writer); with race checks
// the owner reports WW, and the thread the X16 rule names tid_a reports RW.

__device__ PG_RC_INLINE u32 pg_race_check(u32 round, u32 step, u32 tlin, u32 gtid, PgCold& c, u32 evm, u32 val,
                                          u32 site, u32 rec, u32 flat, u32 own, u32 wmax, u32 has_readers, u32 rmin,
                                          u32 rmax) {
    const u32 base = gtid - tlin;
    const u32 w0 = own & 0xFFFu, w1 = wmax & 0xFFFu;
    if (w1 != w0 && tlin == w0) evm |= pg_event(c, evm, PGK_WW, round, rec, flat, gtid, base + w1, site, val, 0);
    if (has_readers && (rmax >> 12) == step) {
        const u32 r0 = rmin & 0xFFFu, r1 = rmax & 0xFFFu;
        if (!(r0 == r1 && w0 == w1 && r0 == w0)) {
            u32 ta, tb;
            if (r0 != w0) { ta = w0; tb = r0; }
            else if (r1 != w0) { ta = w0; tb = r1; }
            else { ta = w1; tb = r0; }
            if (tlin == ta) evm |= pg_event(c, evm, PGK_RW, round, rec, flat, base + ta, base + tb, site, val, 0);
        }
    }
    return evm;
}

template <int A, bool RD>
__device__ __forceinline__ void pg_check_sh(const PgC& C, PgT& t, PgCold& c, u32 flat, u32 val, u32 site) {
    if (PG_T == 1u) {
        pg_sh(t, PG_SH(A, s_own))[flat] = pg_stamp_min(C, t);
        pg_sh(t, PG_SH(A, s_val))[flat] = val;
        return;
    }
    // (thread-private stores: the writer owns its cell, no claim was made)
    const u32 own = PG_TP(A) ? pg_stamp_min(C, t) : pg_sh(t, PG_CAS ? PG_SH(A, s_clm) : PG_SH(A, s_own))[flat];
    if (own == pg_stamp_min(C, t)) {
        pg_sh(t, PG_SH(A, s_val))[flat] = val;
        if (PG_CAS || PG_TP(A)) pg_sh(t, PG_SH(A, s_own))[flat] = own;
    }
#if PG_RACECHK
    if (PG_T > 1u) {
        const u32 wmax = PG_TP(A) ? pg_stamp_max(C, t) : pg_sh(t, PG_SH(A, s_wmax))[flat];
        const u32 rmin = RD ? pg_sh(t, PG_SH(A, s_rmin))[flat] : 0u;
        const u32 rmax = RD ? pg_sh(t, PG_SH(A, s_rmax))[flat] : 0u;
        // (a cell only its writer read this round is no RW race: skip the slow path)
        if ((wmax & 0xFFFu) != (own & 0xFFFu) ||
            (RD && (rmax >> 12) == C.step && (((rmin ^ own) | (rmax ^ own)) & 0xFFFu)))
            t.evm = pg_race_check(C.round, C.step, t.tlin, t.gtid, c, t.evm, val, site, PG_ARR(A).rec_id, flat, own,
                                  wmax, RD, rmin, rmax);
    }
#endif
}

template <int A, bool RD>
__device__ __forceinline__ void pg_check_gt(const PgC& C, PgT& t, PgCold& c, u32 flat, u32 val, u32 site) {
    if (PG_T == 1u) {
        pg_gown<A>(t)[flat] = pg_stamp_min(C, t);
        t.arena[PG_ARR(A).off_val + flat] = val;
        t.arena[PG_ARR(A).off_lw + flat] = t.gtid + 1u;
        return;
    }
    const u32 own = pg_gown<A>(t)[flat];
    if (own == pg_stamp_min(C, t)) {
        t.arena[PG_ARR(A).off_val + flat] = val;
        t.arena[PG_ARR(A).off_lw + flat] = t.gtid + 1u;
    }
#if PG_RACECHK
    if (PG_T > 1u) {
        const u32 wmax = pg_gwmax<A>(t)[flat];
        const u32 rmin = RD ? pg_grmin<A>(t)[flat] : 0u;
        const u32 rmax = RD ? pg_grmax<A>(t)[flat] : 0u;
        // (a cell only its writer read this round is no RW race: skip the slow path)
        if ((wmax & 0xFFFu) != (own & 0xFFFu) ||
            (RD && (rmax >> 12) == C.step && (((rmin ^ own) | (rmax ^ own)) & 0xFFFu)))
            t.evm = pg_race_check(C.round, C.step, t.tlin, t.gtid, c, t.evm, val, site, PG_ARR(A).rec_id, flat, own,
                                  wmax, RD, rmin, rmax);
    }
#endif
}

#if PG_VCLIT
// VC-literal history: this thread's logged writes of the round (every real thread writes its
// count, 0 when it wrote nothing or has exited)
__device__ __forceinline__ void pg_hist_put(const PgC& C, const PgT& t, const PgCold& c) {
    if (t.ekey == 63u || t.blk >= pg_sW.blk1 || C.round >= PG_HIST_R) return;
    u32* e = t.arena + pg_sL.off_hist + (((u64)t.blk * PG_HIST_R + C.round) * PG_T + t.tlin) * (1u + (u32)PG_WMAX);
    e[0] = t.nlog;
    if (t.nlog) e[1] = t.l0cell;
    for (u32 i = 1; i < t.nlog; i++) e[1 + i] = c.lcell[i];
}
#endif

template <class K>
__device__ __forceinline__ void pg_claim_all(const PgC& C, const PgT& t, const PgCold& c) {
    // a 1-thread block is the only writer of its cells in the round (other blocks sharing a
    // global cell are an XB race and re-run sequentially): the check commits directly
    if (t.nlog == 0u || PG_T == 1u || PG_CAS) return;   // (PG_CAS: claimed at store time)
    K::claim_one(C, t, t.l0cell);
    for (u32 i = 1; i < t.nlog; i++) K::claim_one(C, t, c.lcell[i]);
}
template <class K>
__device__ __forceinline__ void pg_check_all(const PgC& C, PgT& t, PgCold& c) {
    if (t.nlog == 0u) return;
#if PG_MSX
    K::check_one(C, t, c, t.l0cell, t.l0v, t.l0site);
    for (u32 i = 1; i < t.nlog; i++) K::check_one(C, t, c, c.lcell[i], c.lvs[i], c.lsite[i]);
#else
    K::check_one(C, t, c, t.l0cell, t.l0val, t.l0site);
    for (u32 i = 1; i < t.nlog; i++) K::check_one(C, t, c, c.lcell[i], c.lval[i], c.lsite[i]);
#endif
}

#if PG_LOCKSTEP
// X25: after the round's commits, every thread of a (real) block copies its share of
// each matched shared array into the instance's snapshot table.
__device__ __noinline__ void pg_snapshot(const PgC& C, const PgT& t) {
    if (t.ekey == 63u || t.blk >= pg_sW.blk1 || C.round >= PG_LOCK_R) return;
    for (u32 a = 0; a < pg_sL.n_arrays; a++) {
        const PgArr& R = pg_sL.arr[a];
        if (R.kind != PGA_SH || R.off_snap == ~0ull) continue;
        const u32* own = (const u32*)(pg_dsmem + t.sg + R.s_own);
        const u32* val = (const u32*)(pg_dsmem + t.sg + R.s_val);
        u32* dst = t.arena + R.off_snap + ((u64)t.blk * PG_LOCK_R + C.round) * R.size * 2u;
        for (u32 i = t.tlin; i < R.size; i += PG_T) {
            const u32 w = pg_owner_step(own[i]) >= C.step0;
            dst[2u * i] = w ? val[i] : 0u;
            dst[2u * i + 1u] = w;
        }
    }
}
#endif

// X19: a block runs rounds 0..0xFFFD; threads still live at round 0xFFFE (the round field
// of X16 keys has 16 bits, 0xFFFF marks MISMATCH / XB) stop with a LIMIT event (val_a 3).
#define PG_ROUND_LIMIT 0xFFFEu
__device__ __forceinline__ void pg_round_limit(const PgC& C, PgT& t, PgCold& c) {
    if (C.round >= PG_ROUND_LIMIT && t.live) {
        PG_EVENT(t, c, PGK_LIMIT, PG_ROUND_LIMIT, PG_NEVER, 0u, t.gtid, PG_NEVER, PG_NEVER, 3u, 0u);
        t.live = 0u;
    }
}

// End of a round when the rounds of a block run inline (K::run, one emulated thread
// per lane): barrier, claims, barrier, checks, then the early-exit vote.  Unless LAST,
// begin the next round and return whether any thread of the CTA is still live.
template <class K, bool LAST>
__device__ __forceinline__ bool pg_round_end(PgC& C, PgT& t, PgCold& c, u32& alive_rounds) {
    const bool warp_blocks = PG_T <= 32u;
#if PG_FAST
    // stores committed in place: one barrier (with the early-exit vote) ends the round;
    // once some thread flagged a race the item stops (every instance of the warp / CTA is
    // re-run exactly, so finishing it would be wasted work)
    C.round++;
    pg_round_limit(C, t, c);
    if (warp_blocks) __syncwarp();
    if (LAST) {
        if (!warp_blocks) __syncthreads();
        pg_fcheck_all<K>(C, t, c);
        return false;
    }
    int more;
    if (warp_blocks) {
        more = __any_sync(PG_FULL, t.live);
        C.abort = __any_sync(PG_FULL, t.fl);
    } else {
        if (t.fl) pg_sAbort = 1u;
        more = __syncthreads_or((int)t.live);
        C.abort = pg_sAbort;
    }
    if (C.abort) {
        t.fl = 1u;
        return false;
    }
    pg_fcheck_all<K>(C, t, c);   // (flags found here stop the item at the next round end)
    if (!more) return false;
    pg_set_step(C, C.step + 1u);
    C.ufuel = 0;
    t.nlog = 0;
    t.fuel = 0;
    alive_rounds += t.live;
    return true;
#else
    if (warp_blocks) __syncwarp(); else __syncthreads();
#if !PG_CAS
    pg_claim_all<K>(C, t, c);
    if (warp_blocks) __syncwarp(); else __syncthreads();
#endif
    pg_check_all<K>(C, t, c);
#if PG_VCLIT
    pg_hist_put(C, t, c);
#endif
#if PG_LOCKSTEP
    if (warp_blocks) __syncwarp(); else __syncthreads();
    pg_snapshot(C, t);
#endif
    C.round++;
    pg_round_limit(C, t, c);
    if (LAST) return false;
    const int more = warp_blocks ? __any_sync(PG_FULL, t.live) : __syncthreads_or((int)t.live);
    if (!more) return false;
    pg_set_step(C, C.step + 1u);
    C.ufuel = 0;
    t.nlog = 0;
    t.fuel = 0;
    alive_rounds += t.live;
    return true;
#endif
}

// ------------------------------------------------------------------ records (H8)
// Each thread keeps its minimum event per kind.  At the end of the CTA: (1) the
// lanes of a warp that belong to the same instance merge (lexicographic min by
// successive warp-wide minima, counts by warp sum); (2) warp leaders deposit
// their results in shared memory and warp 0 merges entries of the same slot;
// (3) one lane per (instance, kind) updates the global slot under its lock.
// All threads of the CTA call pg_flush_cta.
struct PgFlushEntry {
    u64 slot;       // ~0: empty
    u32 cnt;
    u32 f[8];
};

__device__ __forceinline__ void pg_warp_merge(u32 pending, u64 key, u32 cnt_in, const u32* f_in, u32 lane,
                                              u32& leader_out, u64& key_out, u32& cnt_out, u32* best, u32& members) {
    const u32 pm = __ballot_sync(PG_FULL, pending);
    const u32 leader = (u32)__ffs(pm) - 1u;
    const u64 lkey = __shfl_sync(PG_FULL, key, leader);
    u32 cand = pending && key == lkey;
    members = __ballot_sync(PG_FULL, cand);
    cnt_out = __reduce_add_sync(PG_FULL, cand ? cnt_in : 0u);
#pragma unroll
    for (int f = 0; f < 8; f++) {
        best[f] = __reduce_min_sync(PG_FULL, cand ? f_in[f] : PG_NEVER);
        cand = cand && f_in[f] == best[f];
    }
    leader_out = leader;
    key_out = lkey;
}

// true when the slot already holds an event that precedes every event packing to `best`
__device__ __forceinline__ bool pg_slot_skip(PgSlot* s, const u32* best) {
    const u64 pk = ~pg_pack(best);
    if (pk < *(volatile u64*)&s->pkey) return true;   // (pkey only grows: a stale read is safe)
    atomicMax(&s->pkey, pk);
    return false;
}

__device__ __noinline__ void pg_slot_update(PgSlot* s, u32 cnt, const u32* best) {
    atomicAdd(&s->count, (u64)cnt);
    if (pg_slot_skip(s, best)) return;
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

// kmask: the kinds some thread of the CTA recorded (CTA-uniform, from the caller)
__device__ __noinline__ void pg_flush_cta(const PgParams& P, u32 lane, u32 warp, PgCold& c, u32 evm, u32 valid,
                                          u64 slot0, PgFlushEntry* sh /* [32] in shared memory */, u32 kmask,
                                          u32 seed_s = 0) {
    const u32 nwarps = blockDim.x >> 5;
    for (u32 k = 0; k < PG_NK; k++) {
        if (!((kmask >> k) & 1u)) continue;
        if (lane == 0) sh[warp].slot = ~0ull;
        __syncwarp();
        u32 pending = valid && ((evm >> k) & 1u);
        bool first = true;
        for (;;) {
            if (!__any_sync(PG_FULL, pending)) break;
            u32 leader, cnt, members, best[8];
            u64 key;
            u32 f_in[8];
#pragma unroll
            for (int i = 0; i < 8; i++) f_in[i] = pending ? c.ebest[k][i] : PG_NEVER;
#if PG_MSX
            f_in[6] = pending ? c.ebv[k][seed_s] : PG_NEVER;   // (multi-seed exact pass: this seed's values)
            f_in[7] = pending ? ((c.vbx >> k) & 1u ? c.ebvs[k][seed_s] : c.ebvb[k]) : PG_NEVER;
#endif
            pg_warp_merge(pending, slot0, pending ? c.ecnt[k] : 0u, f_in, lane, leader, key, cnt, best, members);
            if (lane == leader) {
                if (first) {   // the common case: one instance per warp -> deposit for the CTA merge
                    sh[warp].slot = key;
                    sh[warp].cnt = cnt;
#pragma unroll
                    for (int i = 0; i < 8; i++) sh[warp].f[i] = best[i];
                } else {
                    pg_slot_update(P.slots + key + k, cnt, best);
                }
            }
            first = false;
            if (members & (1u << lane)) pending = 0u;
            __syncwarp();
        }
        __syncthreads();
        if (warp == 0) {
            const bool has = lane < nwarps && sh[lane].slot != ~0ull;
            u32 pend = has;
            const u64 skey = has ? sh[lane].slot : 0ull;
            const u32 scnt = has ? sh[lane].cnt : 0u;
            u32 sf[8];
#pragma unroll
            for (int i = 0; i < 8; i++) sf[i] = has ? sh[lane].f[i] : PG_NEVER;
            for (;;) {
                if (!__any_sync(PG_FULL, pend)) break;
                u32 leader, cnt, members, best[8];
                u64 key;
                pg_warp_merge(pend, skey, scnt, sf, lane, leader, key, cnt, best, members);
                if (lane == leader) pg_slot_update(P.slots + key + k, cnt, best);
                if (members & (1u << lane)) pend = 0u;
                __syncwarp();
            }
        }
        __syncthreads();
    }
}

#if PG_MSX
// Record flush of the multi-seed exact pass: every event of this pass carries the recording
// thread's gtid as tid_a (OOB, UNINIT, LIMIT, WW and RW alike), so two candidates never tie
// on the seed-independent fields (round, array, addr, tid_a, tid_b, site); the merge runs
// once per kind on those fields and the winner's per-seed values fill the seeds' slots.  The
// group's first slot's lock guards all of its seeds' slots (always updated together).
struct PgFlushEntryMs {
    u64 slot;       // ~0: empty
    u32 cnt, nsv;
    u32 f[6];
    u32 v[PG_MS][2];
};
__device__ __noinline__ void pg_slot_update_ms(PgSlot* s0, u64 step, u32 nsv, u32 cnt, const u32* f6,
                                               const u32 (*v)[2]) {
    for (u32 q = 0; q < nsv; q++) atomicAdd(&s0[q * step].count, (u64)cnt);
    if (pg_slot_skip(s0, f6)) return;
    while (atomicCAS(&s0->lock, 0u, 1u) != 0u) {
    }
    __threadfence();
    volatile PgSlot* vs = s0;
    bool less = !vs->has;
    if (!less) {
        for (int i = 0; i < 6; i++) {
            const u32 cur = vs->f[i];
            if (f6[i] != cur) {
                less = f6[i] < cur;
                break;
            }
        }
    }
    if (less) {
        for (u32 q = 0; q < nsv; q++) {
            volatile PgSlot* t = s0 + q * step;
#pragma unroll
            for (int i = 0; i < 6; i++) t->f[i] = f6[i];
            t->f[6] = v[q][0];
            t->f[7] = v[q][1];
            t->has = 1u;
        }
    }
    __threadfence();
    atomicExch(&s0->lock, 0u);
}
__device__ __noinline__ void pg_flush_cta_ms(const PgParams& P, u32 lane, u32 warp, PgCold& c, u32 evm, u32 valid,
                                             u64 slot0, u32 nsv, PgFlushEntryMs* sh /* [32] */, u32 kmask) {
    const u32 nwarps = blockDim.x >> 5;
    const u64 step = pg_sW.slot_step;
    for (u32 k = 0; k < PG_NK; k++) {
        if (!((kmask >> k) & 1u)) continue;
        if (lane == 0) sh[warp].slot = ~0ull;
        __syncwarp();
        u32 pending = valid && ((evm >> k) & 1u);
        bool first = true;
        for (;;) {
            if (!__any_sync(PG_FULL, pending)) break;
            u32 leader, cnt, members, best[8];
            u64 key;
            u32 f_in[8];
#pragma unroll
            for (int i = 0; i < 6; i++) f_in[i] = pending ? c.ebest[k][i] : PG_NEVER;
            f_in[6] = f_in[7] = pending ? 0u : PG_NEVER;
            pg_warp_merge(pending, slot0, pending ? c.ecnt[k] : 0u, f_in, lane, leader, key, cnt, best, members);
            bool same = pending && slot0 == key;
#pragma unroll
            for (int i = 0; i < 6; i++) same = same && f_in[i] == best[i];
            const u32 win = (u32)__ffs(__ballot_sync(PG_FULL, same)) - 1u;
            u32 vv[PG_MS][2];
#pragma unroll
            for (u32 q = 0; q < PG_MS; q++) {
                vv[q][0] = __shfl_sync(PG_FULL, c.ebv[k][q], win);
                vv[q][1] = __shfl_sync(PG_FULL, (c.vbx >> k) & 1u ? c.ebvs[k][q] : c.ebvb[k], win);
            }
            const u32 wn = __shfl_sync(PG_FULL, nsv, win);
            if (lane == leader) {
                if (first) {   // the common case: one group per warp -> deposit for the CTA merge
                    sh[warp].slot = key;
                    sh[warp].cnt = cnt;
                    sh[warp].nsv = wn;
#pragma unroll
                    for (int i = 0; i < 6; i++) sh[warp].f[i] = best[i];
#pragma unroll
                    for (u32 q = 0; q < PG_MS; q++) { sh[warp].v[q][0] = vv[q][0]; sh[warp].v[q][1] = vv[q][1]; }
                } else {
                    pg_slot_update_ms(P.slots + key + k, step, wn, cnt, best, vv);
                }
            }
            first = false;
            if (members & (1u << lane)) pending = 0u;
            __syncwarp();
        }
        __syncthreads();
        if (warp == 0) {
            const bool has = lane < nwarps && sh[lane].slot != ~0ull;
            u32 pend = has;
            const u64 skey = has ? sh[lane].slot : 0ull;
            const u32 scnt = has ? sh[lane].cnt : 0u;
            u32 sf[8];
#pragma unroll
            for (int i = 0; i < 6; i++) sf[i] = has ? sh[lane].f[i] : PG_NEVER;
            sf[6] = sf[7] = has ? 0u : PG_NEVER;
            for (;;) {
                if (!__any_sync(PG_FULL, pend)) break;
                u32 leader, cnt, members, best[8];
                u64 key;
                pg_warp_merge(pend, skey, scnt, sf, lane, leader, key, cnt, best, members);
                bool same = pend && skey == key;
#pragma unroll
                for (int i = 0; i < 6; i++) same = same && sf[i] == best[i];
                const u32 win = (u32)__ffs(__ballot_sync(PG_FULL, same)) - 1u;
                if (lane == leader) pg_slot_update_ms(P.slots + key + k, step, sh[win].nsv, cnt, best, sh[win].v);
                if (members & (1u << lane)) pend = 0u;
                __syncwarp();
            }
        }
        __syncthreads();
    }
}
#endif

// ------------------------------------------------------------------ CTA main loop
// A CTA runs G groups of one launch in lock step.  Group g emulates, for seed
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

#if PG_DIVBAR
// X18 at round end: the barrier sites the live threads of each emulated block wait at.
// Two or more distinct sites -> one BARRIER_DIV event: (lowest site, second-lowest site)
// and the lowest thread waiting at each (gtid), in the order of DESIGN.md X16/X18.
// dv: 4 words per group (s0, s1, t0, t1), all-ones between rounds.
template <class K>
__device__ __forceinline__ void pg_barrier_div(const PgC& C, PgT* T, PgCold* Cd, const u32* rsm, u32 V, u32 g,
                                               u32 tl0, u32 inst_ok, bool warp_blocks, u32* dv_all) {
    u32* dv = dv_all + 4u * (inst_ok ? g : 0u);
    u32 site[PG_VMAX];
#pragma unroll
    for (u32 v = 0; v < PG_VMAX; v++)
        site[v] = (v < V && inst_ok && T[v].live) ? K::sync_site(rsm[v]) : PG_NEVER;
#define PG_DV_BAR() do { if (warp_blocks) __syncwarp(); else __syncthreads(); } while (0)
#pragma unroll
    for (u32 v = 0; v < PG_VMAX; v++)
        if (site[v] != PG_NEVER) atomicMin(&dv[0], site[v]);
    PG_DV_BAR();
    const u32 s0 = inst_ok ? dv[0] : PG_NEVER;
#pragma unroll
    for (u32 v = 0; v < PG_VMAX; v++)
        if (site[v] != PG_NEVER && site[v] != s0) atomicMin(&dv[1], site[v]);
    PG_DV_BAR();
    const u32 s1 = inst_ok ? dv[1] : PG_NEVER;
    if (s1 != PG_NEVER) {
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++) {
            if (site[v] == s0) atomicMin(&dv[2], T[v].gtid);
            else if (site[v] == s1) atomicMin(&dv[3], T[v].gtid);
        }
    }
    PG_DV_BAR();
    if (s1 != PG_NEVER && tl0 == 0u) PG_EVENT(T[0], Cd[0], PGK_BARRIER_DIV, C.round, PG_NEVER, 0u, dv[2], dv[3], s0, s1, 0u);
    PG_DV_BAR();
    if (inst_ok && tl0 == 0u) dv[0] = dv[1] = dv[2] = dv[3] = PG_NEVER;
    PG_DV_BAR();
#undef PG_DV_BAR
}
#endif

// The launch descriptor (the IR's layout constants: array offsets, sizes, strides, 2.3 KB)
// of the item is staged into shared memory by the TMA engine: one thread arms the CTA's
// mbarrier with the byte count and issues a 1-D cp.async.bulk; every thread waits on the
// barrier's phase (one phase per item).
__device__ __forceinline__ u32 pg_smem_addr(const void* p) { return (u32)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void pg_desc_bulk_issue(const PgLaunchK* src) {
    const u32 bar = pg_smem_addr(&pg_sBar), dst = pg_smem_addr(&pg_sL), bytes = (u32)sizeof(PgLaunchK);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // (earlier generic reads of pg_sL)
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ void pg_desc_bulk_wait(u32 phase) {
    const u32 bar = pg_smem_addr(&pg_sBar);
    u32 done = 0;
    while (!done)
        asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                     : "=r"(done) : "r"(bar), "r"(phase) : "memory");
}

template <class K>
__device__ __forceinline__ void pg_item(const PgParams& P, const u32 wi, u32& phase) {
    __shared__ u32 s_flag;
    // (launches the sequential pass takes whole this check: nothing to do in the parallel passes)
    if (P.seq != 1u && P.seq_pref && P.seq_pref[P.work[wi].launch]) return;
    if (P.seq) {
        // re-runs: only items with a flagged instance (seq 1: a global cell shared between
        // blocks; seq 2: a race the optimistic pass flagged)
        if (threadIdx.x == 0) {
            const PgWork& w = P.work[wi];
            u32 f = 0;
            for (u32 i = 0; i < w.nseeds; i++) f |= P.xb_flag[w.inst0 + i];
            s_flag = f;
        }
        __syncthreads();
        if (!s_flag) return;
    }
    {
        if (threadIdx.x == 0) pg_desc_bulk_issue(&P.launches[P.work[wi].launch]);
        const u32* ws = (const u32*)&P.work[wi];
        u32* wd = (u32*)&pg_sW;
        for (u32 i = threadIdx.x; i < sizeof(PgWork) / 4; i += blockDim.x) wd[i] = ws[i];
        pg_desc_bulk_wait(phase);
        phase ^= 1u;
    }
#if PG_DATAFLOW
    if (threadIdx.x == 0) pg_sDf = PgDf{P.df_rows, P.df_count, P.seed_base, P.df_cap};
#endif
    __syncthreads();
    const u32 G = pg_sW.ngroups, GB = pg_sW.gb;
    if (P.seq == 1u) {
        // fresh arenas and slots for every seed of the group (the parallel pass is discarded)
        for (u32 ms = 0; ms < pg_sW.nseeds; ms++) {
            const u64 seed = P.seed_base + (u64)(pg_sW.seed_j0 + ms * pg_sW.seed_jstep);
            u32* ar = P.arena + pg_sW.arena_off + (u64)ms * pg_sL.arena_stride;
            for (u32 a = 0; a < pg_sL.n_arrays; a++) {
                const PgArr& R = pg_sL.arr[a];
                if (R.kind != PGA_GT) continue;
                for (u32 i = threadIdx.x; i < R.size; i += blockDim.x) {
                    if (!P.keep_vals) ar[R.off_val + i] = pg_init_value(P, seed, R.gid, i);
                    ar[R.off_own + i] = PG_NEVER;
                    ar[R.off_lw + i] = 0u;
                    if (R.off_wmax != ~0ull) ar[R.off_wmax + i] = 0u;
                    for (u32 q = 0; q < R.rsets; q++) {
                        if (R.off_rmin != ~0ull) ar[R.off_rmin + (u64)q * R.size + i] = PG_NEVER;
                        if (R.off_rmax != ~0ull) ar[R.off_rmax + (u64)q * R.size + i] = 0u;
                    }
                    if (R.off_xf != ~0ull) { ar[R.off_xf + i] = PG_NEVER; ar[R.off_xl + i] = 0u; }
                }
            }
            if (threadIdx.x < PG_NK) {
                PgSlot* sl = P.slots + pg_sW.slot0 + (u64)ms * pg_sW.slot_step + threadIdx.x;
                sl->count = 0;
                sl->has = 0;
                sl->lock = 0;
                sl->pkey = 0;
            }
            if (threadIdx.x == 0u) P.inst_cnt[pg_sW.inst0 + ms] = 0ull;   // counted again below
#if PG_OPCOUNT
            if (threadIdx.x == 0u) P.op_cnt[pg_sW.inst0 + ms] = 0ull;
#endif
        }
        __threadfence();
        __syncthreads();
    }
    const u32 gbytes = PG_GBYTES;
    const u32 T_ = PG_T;
    const bool warp_blocks = T_ <= 32u;  // an emulated block never spans warps: warp-level barriers suffice
    u64* sstats = (u64*)(pg_dsmem + (u64)PG_PK * gbytes);
    u32* s_grounds = (u32*)(sstats + ((PG_BANKCHK || PG_COALCHK) ? PG_NSTATS * 8 : 0));  // per group (T > 32)
    // shared regions: initialised once per CTA (stamps are step-tagged)
    {
        const u32 zw = (PG_NOFF - PG_ZOFF) / 4u;
        const u32 nw = (gbytes - PG_NOFF) / 4u;
        const u32 per = zw + nw;
        for (u32 i = threadIdx.x; i < G * per; i += blockDim.x) {
            const u32 gi = i / per, j = i - gi * per;
            u32* base = (u32*)(pg_dsmem + (u64)gi * gbytes + PG_ZOFF);
            base[j] = j < zw ? 0u : PG_NEVER;
        }
    }
#if PG_BANKCHK || PG_COALCHK
    for (u32 i = threadIdx.x; i < PG_NSTATS * 8; i += blockDim.x) sstats[i] = 0;
#else
    sstats = nullptr;
#endif
    for (u32 i = threadIdx.x; i < PG_PK; i += blockDim.x) s_grounds[i] = 0;
#if PG_DIVBAR
    for (u32 i = threadIdx.x; i < 4u * PG_PK; i += blockDim.x) s_grounds[PG_PK + i] = PG_NEVER;
#endif

    PgC C;
    pg_set_step(C, 0u);
    C.abort = 0;
#if PG_FAST
    if (threadIdx.x == 0) pg_sAbort = 0u;   // (published by the barrier below)
#endif
    C.fuel = P.fuel;
    const u32 lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
    u32 g, tl0, lane_ok, ekey;
    if (warp_blocks) {
        const u32 sub = lane / T_;
        g = warp * PG_GPW + sub;
        tl0 = lane - sub * T_;
        lane_ok = sub < PG_GPW;
        ekey = lane_ok ? sub : 63u;
    } else {
        g = warp / PG_WPG;
        tl0 = (warp % PG_WPG) * 32u + lane;
        lane_ok = 1u;
        ekey = 0u;
    }
    // (exact re-run, P.seq == 2: only the instances the optimistic pass flagged)
    const u32 inst_ok = lane_ok && g < G && (P.seq != 2u || P.xb_flag[pg_sW.inst0 + (g / GB) * PG_MS] != 0u);
    const u32 gc = inst_ok ? g : 0u;
    const u32 ms = gc / GB, bs = gc % GB;
    const u32 sb = ms * PG_MS;   // the group's first seed within the item (multi-seed lanes: PG_MS seeds)
    const u32 nsv = PG_MS > 1 ? min((u32)PG_MS, pg_sW.nseeds - min(sb, pg_sW.nseeds)) : 1u;
    typename K::Frame F[PG_VMAX];
    PgT T[PG_VMAX];
    PgCold Cd[PG_VMAX];
    const u32 V = PG_VMAX > 1 ? PG_VV : 1u;
#pragma unroll
    for (u32 v = 0; v < PG_VMAX; v++) {
        if (v >= V) break;
        PgT& t = T[v];
        t.tlin = tl0 + v * (32u * PG_WPG);   // virtual thread v: lanes of the v-th slice of the block
        const u32 ok = inst_ok && t.tlin < T_;
        t.ekey = ok ? ekey : 63u;
        t.lane = lane;
        t.tid[0] = t.tlin % PG_BDIM0;
        t.tid[1] = (t.tlin / PG_BDIM0) % PG_BDIM1;
        t.tid[2] = t.tlin / (PG_BDIM0 * PG_BDIM1);
        t.seed = P.seed_base + (u64)(pg_sW.seed_j0 + sb * pg_sW.seed_jstep);
        t.arena = P.arena + pg_sW.arena_off + (u64)sb * pg_sL.arena_stride;
        t.input = P.input + pg_sW.input_off + (u64)sb * pg_sL.input_stride;
        t.nsv = nsv;
        t.sg = gc * gbytes;
        t.l0cell = t.l0val = t.l0site = 0u;
        t.evm = 0u;
        t.fl = 0u;
        t.live = ok;
#if PG_OPCOUNT
        t.ops = 0u;
#endif
    }
    __syncthreads();
    const bool grid_1d = pg_sL.gdim[1] == 1u && pg_sL.gdim[2] == 1u;
    const bool grid_pow2 = !(pg_sL.gdim[0] & (pg_sL.gdim[0] - 1u)) && !(pg_sL.gdim[1] & (pg_sL.gdim[1] - 1u));
    const u32 gsh0 = __ffs(pg_sL.gdim[0]) - 1, gsh1 = __ffs(pg_sL.gdim[1]) - 1;
    u64 inst = 0;  // instances of this group (accumulated by its lane tl0 == 0)
    const u32 nsteps = (pg_sW.blk1 - pg_sW.blk0 + GB - 1) / GB;
    for (u32 st = 0; st < nsteps; st++) {
        const u32 blk = pg_sW.blk0 + st * GB + bs;
        const u32 blk_ok = blk < pg_sW.blk1;
        pg_set_step0(C, C.step + 1u);
        u32 alive_rounds = 0;  // rounds this thread entered alive (X19: group rounds = max over threads)
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++) {
            if (v >= V) break;
            PgT& t = T[v];
            t.blk = blk;
            if (grid_1d) {
                t.bid[0] = blk;
                t.bid[1] = t.bid[2] = 0u;
            } else if (grid_pow2) {   // (power-of-two grid dims: shifts instead of divisions)
                t.bid[0] = blk & (pg_sL.gdim[0] - 1u);
                t.bid[1] = (blk >> gsh0) & (pg_sL.gdim[1] - 1u);
                t.bid[2] = blk >> (gsh0 + gsh1);
            } else {   // (blk < 2^20: division by multiply-high with the launch's magic numbers)
                const u32 q0 = (u32)(((u64)blk * pg_sL.gmag0) >> 40);
                const u32 q01 = (u32)(((u64)blk * pg_sL.gmag01) >> 40);
                t.bid[0] = blk - q0 * pg_sL.gdim[0];
                t.bid[1] = q0 - q01 * pg_sL.gdim[1];
                t.bid[2] = q01;
            }
            t.live = inst_ok && t.tlin < T_ && blk_ok;
            t.gtid = blk * T_ + t.tlin;
            K::init(F[v], C, t);
        }
#if PG_DATAFLOW
        if (pg_sL.off_step0 != ~0ull && inst_ok && tl0 == 0u && blk_ok) T[0].arena[pg_sL.off_step0 + blk] = C.step0;
#endif
        C.round = 0;
#if PG_VMAX == 1 && !PG_DIVBAR
        {   // rounds inline: K::run ends each round at its barrier (pg_round_end)
            PgT& t = T[0];
            pg_set_step(C, C.step + 1u);
            C.ufuel = 0;
            t.nlog = 0;
            t.fuel = 0;
            alive_rounds = t.live;
            K::run(F[0], C, t, Cd[0], sstats, alive_rounds);
#if PG_VCLIT
            if (inst_ok && tl0 == 0u && blk_ok) t.arena[pg_sL.off_hround + blk] = C.round;
#endif
        }
#else
        u32 resume = 0;
#if PG_DIVBAR
        u32 rsm[PG_VMAX];   // per-thread resume points: each thread resumes after its own barrier (X18)
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++) rsm[v] = 0u;
#endif
        for (;;) {
            pg_set_step(C, C.step + 1u);
            C.ufuel = 0;
            u32 r = PG_END;
            u32 any_start = 0;
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                any_start |= T[v].live;
                T[v].nlog = 0;
                T[v].fuel = 0;
#if PG_DIVBAR
                if (T[v].live) rsm[v] = K::seg(F[v], C, T[v], Cd[v], sstats, rsm[v]);
#else
                r = K::seg(F[v], C, T[v], Cd[v], sstats, resume);
#endif
            }
            alive_rounds += any_start;
#if PG_DIVBAR
            pg_barrier_div<K>(C, T, Cd, rsm, V, g, tl0, inst_ok, warp_blocks, s_grounds + PG_PK);
#endif
            u32 any = 0;
#if PG_FAST
            if (warp_blocks) __syncwarp();
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                any |= T[v].live;
            }
#else
            if (warp_blocks) __syncwarp(); else __syncthreads();
#if !PG_CAS
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                pg_claim_all<K>(C, T[v], Cd[v]);
            }
            if (warp_blocks) __syncwarp(); else __syncthreads();
#endif
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                pg_check_all<K>(C, T[v], Cd[v]);
                any |= T[v].live;
            }
#endif
            C.round++;
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++)
                if (v < V) pg_round_limit(C, T[v], Cd[v]);
#if PG_FAST
            u32 fl = 0;
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                fl |= T[v].fl;
            }
            int more;
            if (warp_blocks) {
                more = __any_sync(PG_FULL, any);
                C.abort = __any_sync(PG_FULL, fl);
            } else {
                if (fl) pg_sAbort = 1u;
                more = __syncthreads_or((int)any);
                C.abort = pg_sAbort;
            }
            if (C.abort) {
#pragma unroll
                for (u32 v = 0; v < PG_VMAX; v++) T[v].fl = 1u;
                break;
            }
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
                pg_fcheck_all<K>(C, T[v], Cd[v]);
            }
#else
            const int more = warp_blocks ? __any_sync(PG_FULL, any) : __syncthreads_or((int)any);
#endif
#if PG_DIVBAR
            if (!more) break;
#else
            if (r == PG_END || !more) break;
#endif
            resume = r;
        }
#endif
        // rounds of this group's block = max over its threads of the rounds they entered alive
        u32 grounds;
        if (warp_blocks && (T_ & (T_ - 1u)) == 0u) {
            // groups are aligned power-of-two lane segments: butterfly max (no per-group masks,
            // which would serialise the warp once per group)
            grounds = alive_rounds;
            for (u32 o = 1u; o < T_; o <<= 1) grounds = max(grounds, __shfl_xor_sync(PG_FULL, grounds, o));
        } else if (warp_blocks) {
            if (inst_ok && alive_rounds) atomicMax(&s_grounds[g], alive_rounds);
            __syncwarp();
            grounds = inst_ok ? s_grounds[g] : 0u;
            __syncwarp();
            if (inst_ok && tl0 == 0u) s_grounds[g] = 0u;
            __syncwarp();
        } else {   // a warp lies in one group: warp max, then one shared atomic per warp
            const u32 wm = __reduce_max_sync(PG_FULL, inst_ok ? alive_rounds : 0u);
            if (lane == 0u && inst_ok && wm) atomicMax(&s_grounds[g], wm);
            __syncthreads();
            grounds = inst_ok ? s_grounds[g] : 0u;
            __syncthreads();
            if (inst_ok && tl0 == 0u) s_grounds[g] = 0u;
        }
        inst += (u64)T_ * grounds;
        if (C.abort) break;   // (PG_FAST; warp- or CTA-uniform like the barriers above)
    }
    __syncthreads();
#if PG_RACECHK
    // X4: cross-block races on global cells written by this kernel (sequential pass: the
    // CTA owns whole instances; the parallel pass leaves them to the flagged re-run)
    if (P.seq == 1u && pg_sL.nblocks > 1) {
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++) {
            if (v >= V) break;
            PgT& t = T[v];
            if (!(inst_ok && t.tlin < T_)) continue;
            for (u32 a = 0; a < pg_sL.n_arrays; a++) {
                const PgArr& ar = pg_sL.arr[a];
                if (ar.kind != PGA_GT || ar.off_xf == ~0ull) continue;
                const u32* xf = t.arena + ar.off_xf;
                const u32* xl = t.arena + ar.off_xl;
                const u32* lw = t.arena + ar.off_lw;
                const u32* val = t.arena + ar.off_val;
                for (u32 i = t.tlin; i < ar.size; i += T_)
                    if (lw[i] && xf[i] != xl[i])
                        PG_EVENT(t, Cd[v], PGK_XB, 0xFFFFu, ar.rec_id, i, xf[i] - 1u, xl[i] - 1u, PG_NEVER, val[i], 0u);
            }
            // (the sequential preference of the next check counts instances that raced here)
            if ((t.evm >> PGK_XB) & 1u) P.xb_flag[pg_sW.inst0 + sb] = 2u;
        }
    }
#endif
    {
        __shared__ PgFlushEntry s_flush[32];
        u32 any_ev = 0;
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++) {
            if (v >= V) break;
            any_ev |= T[v].evm;
        }
        // the kinds recorded anywhere in the CTA: one barrier, then only those kinds are merged
        __shared__ u32 s_kmask;
        if (threadIdx.x == 0) s_kmask = 0u;
        __syncthreads();
        {
            const u32 wm = __reduce_or_sync(PG_FULL, inst_ok ? any_ev : 0u);
            if (lane == 0u && wm) atomicOr(&s_kmask, wm);
        }
        __syncthreads();
        const u32 kmask = s_kmask;
        if (kmask) {
#pragma unroll
            for (u32 v = 0; v < PG_VMAX; v++) {
                if (v >= V) break;
#if PG_MSX
                __shared__ PgFlushEntryMs s_flush_ms[32];
                pg_flush_cta_ms(P, lane, warp, Cd[v], T[v].evm, inst_ok && T[v].tlin < T_,
                                pg_sW.slot0 + (u64)sb * pg_sW.slot_step, nsv, s_flush_ms, kmask);
#else
                pg_flush_cta(P, lane, warp, Cd[v], T[v].evm, inst_ok && T[v].tlin < T_, pg_sW.slot0 + (u64)sb * pg_sW.slot_step,
                             s_flush, kmask);
#endif
            }
        }
    }
#if PG_FAST
    {   // flag instances with a possible race for the exact re-run
        u32 fl = 0;
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++) {
            if (v >= V) break;
            fl |= T[v].fl;
        }
        if (fl && inst_ok)
        {
            for (u32 i = 0; i < nsv; i++) P.xb_flag[pg_sW.inst0 + sb + i] = 1u;
            if (P.flag_any) *P.flag_any = 1u;
        }
    }
#endif
    // instances (X19) per batch-local instance (a re-run replaces its instance's count):
    // one atomic per warp when the warp's groups belong to one instance (block-major packing)
    if (P.count_inst) {
        u64 x = (inst_ok && tl0 == 0u) ? inst : 0ull;
        const u32 key = x ? pg_sW.inst0 + sb : PG_NEVER;
        const u32 k0 = __reduce_min_sync(PG_FULL, key);
        if (__all_sync(PG_FULL, key == PG_NEVER || key == k0)) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) x += __shfl_down_sync(PG_FULL, x, o);
            if (lane == 0u && x) {
                // (multi-seed lanes: every seed of the group ran the same rounds)
                const u32 n0 = PG_MS > 1 ? min((u32)PG_MS, pg_sW.nseeds - (k0 - pg_sW.inst0)) : 1u;
                for (u32 i = 0; i < n0; i++) atomicAdd(&P.inst_cnt[k0 + i], x);
            }
        } else if (x) {
            for (u32 i = 0; i < nsv; i++) atomicAdd(&P.inst_cnt[key + i], x);
        }
    }
#if PG_OPCOUNT
    {   // IR operations per batch-local instance (PG_CHK_OPCOUNT; one seed per group here)
        u64 x = 0;
#pragma unroll
        for (u32 v = 0; v < PG_VMAX; v++)
            if (v < V && inst_ok) x += T[v].ops;
        if (x) atomicAdd(&P.op_cnt[pg_sW.inst0 + sb], x);
    }
#endif
#if PG_BANKCHK || PG_COALCHK
    __syncthreads();
    if (P.site_stats) {
        u64* dst = P.site_stats + (u64)(P.seq == 1u ? pg_sW.launch : pg_sW.item) * P.max_sites * 8u;
        for (u32 i = threadIdx.x; i < PG_NSTATS * 8 && i < P.max_sites * 8; i += blockDim.x) {
            const u32 col = i & 7u;
            if (col == 3) atomicMax(&dst[i], sstats[i]);
            else if (col == 0) { if (sstats[i]) dst[i] = sstats[i]; }
            else if (sstats[i]) atomicAdd(&dst[i], sstats[i]);
        }
    }
#endif
}

// One work item per CTA, or (sequential pass) a grid-stride loop over the items the
// selection kernel listed: a pass with nothing to re-run costs one short launch.
template <class K>
__device__ __forceinline__ void pg_main(const PgParams& P) {
    if (P.seq && P.flag_any && *(volatile const u32*)P.flag_any == 0u) return;   // nothing to re-run
    const bool listed = P.work_count != nullptr;
    const u32 n = listed ? *P.work_count : P.n_work ? P.n_work : blockIdx.x + 1u;
    if (threadIdx.x == 0) {   // the descriptor's mbarrier: one arrival (the issuing thread) per phase
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(pg_smem_addr(&pg_sBar)) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    u32 phase = 0;
    for (u32 i = blockIdx.x; i < n; i += gridDim.x) {   // (one call site: one inlined copy)
        pg_item<K>(P, listed ? P.work_list[i] : i, phase);
        __syncthreads();
    }
}
