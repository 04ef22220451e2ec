// kernels.cu — ahead-of-time CUDA kernels of libpgvc (sm_100a):
//   K1 pg_gen_inputs  : initial global-array contents from the PRF (H2, X7/X8)
//   K3 pg_compare     : comparative assertion o_s = o_t (H7)
//   K4 pg_summarize / pg_scan / pg_compact : canonical record list + counters (H8, X16)
// The evaluation kernel K2 is generated per IR (codegen.cpp) and JIT-compiled.
#include <cuda_runtime.h>
#include <stdint.h>

#include "pg_layout.h"
#include "pg_prf.cuh"

namespace {



// CTA tasks of the per-(job, instance) kernels (K1, K2b, K3): jobs carry task0, the index
// of their first task; a task is a PG_FILL_CHUNK-word chunk of one instance (arrays of more
// than PG_FILL_SMALL words) or 8 instances, a warp each.  Returns the job of `task`.
template <class J>
__device__ __forceinline__ u32 pg_task_job(const J* jobs, u32 n_jobs, u32 task_base, u32 task, u32* s_job) {
    if (threadIdx.x == 0) {
        // a CTA visits its tasks in increasing order, so the job index never decreases:
        // gallop forward from the last job found, then bisect
        u32 lo = *s_job < n_jobs ? *s_job : 0u, hi = lo, d = 1;
        while (hi + 1u < n_jobs && jobs[hi + 1u].task0 - task_base <= task) {
            lo = hi + 1u;
            hi = min(n_jobs - 1u, hi + d);
            d <<= 1;
            if (jobs[hi].task0 - task_base > task) { hi -= 1u; break; }
            lo = hi;
        }
        while (lo < hi) {
            const u32 mid = (lo + hi + 1u) >> 1;
            if (jobs[mid].task0 - task_base <= task) lo = mid;
            else hi = mid - 1u;
        }
        *s_job = lo;
    }
    __syncthreads();
    const u32 j = *s_job;
    __syncthreads();   // (thread 0 rewrites *s_job for the next task)
    return j;
}

// One CTA task per grid-stride step (tasks of all jobs numbered consecutively, task0 per
// job): a 4096-word chunk of one instance stored as 128-bit words, or 8 small instances, a
// warp each.  With `flags`, only flagged instances are (re-)initialised: the exact re-run of
// the instances the optimistic pass flagged.
__device__ __forceinline__ u32 fill_value(u32 op, u32 mode, u32 range, u32 mask, u32 value, u64 key, u64 seed,
                                          u32 i) {
    if (op == PGF_CONST) return value;
    u32 v;
    if (mode == 1) v = i < 64 ? (u32)((seed >> i) & 1ull) : 0u;                 // BITS01
    else if (mode == 2) v = pg_rand32_k(key, i) % (range ? range : 1u);          // RANGE(k)
    else v = pg_rand32_k(key, i);                                               // RAND32
    return v & mask;
}
__global__ void __launch_bounds__(256) pg_gen_inputs(const PgFill* __restrict__ jobs, u32 n_jobs, u32 task_base,
                                                     u32 n_tasks, const PgRegions R, u64 seed_base, u32 mode,
                                                     u32 range, u32 mask, const u32* flags, const u32* any) {
    if (flags && !*any) return;   // re-initialisation with nothing flagged
    __shared__ u32 s_job;
    if (threadIdx.x == 0) s_job = 0u;
    for (u32 task = blockIdx.x; task < n_tasks; task += gridDim.x) {
        const PgFill f = jobs[pg_task_job(jobs, n_jobs, task_base, task, &s_job)];
        const u32 lt = task - (f.task0 - task_base);
        u32* region = R.r[f.target];
        if (f.n > PG_FILL_SMALL) {
            const u32 nch = (f.n + PG_FILL_CHUNK - 1u) / PG_FILL_CHUNK;
            const u32 inst = lt / nch, w0 = (lt - inst * nch) * PG_FILL_CHUNK;
            const u32 w1 = min(f.n, w0 + PG_FILL_CHUNK);
            const u32 ai = inst * f.istep;
            if (flags && !flags[f.inst0 + ai]) continue;
            u32* base = region + f.dst + (u64)ai * f.stride;   // (128-byte aligned: arena layout)
            const u64 seed = seed_base + (u64)f.j0 + (u64)ai * f.jstep;
            const u64 key = pg_sm64(seed) ^ ((u64)f.gid << 48);
            const u32 w4 = w0 + ((w1 - w0) & ~3u);
            for (u32 i = w0 + 4u * threadIdx.x; i < w4; i += 4u * blockDim.x) {
                uint4 q;
                q.x = fill_value(f.op, mode, range, mask, f.value, key, seed, i);
                q.y = fill_value(f.op, mode, range, mask, f.value, key, seed, i + 1u);
                q.z = fill_value(f.op, mode, range, mask, f.value, key, seed, i + 2u);
                q.w = fill_value(f.op, mode, range, mask, f.value, key, seed, i + 3u);
                *(uint4*)(base + i) = q;
            }
            for (u32 i = w4 + threadIdx.x; i < w1; i += blockDim.x)
                base[i] = fill_value(f.op, mode, range, mask, f.value, key, seed, i);
        } else {
            const u32 inst = lt * 8u + (threadIdx.x >> 5), lane = threadIdx.x & 31u;
            const u32 ai = inst * f.istep;
            if (inst >= f.n_inst || (flags && !flags[f.inst0 + ai])) continue;
            u32* base = region + f.dst + (u64)ai * f.stride;
            const u64 seed = seed_base + (u64)f.j0 + (u64)ai * f.jstep;
            const u64 key = pg_sm64(seed) ^ ((u64)f.gid << 48);
            for (u32 i = lane; i < f.n; i += 32u) base[i] = fill_value(f.op, mode, range, mask, f.value, key, seed, i);
        }
    }
}

// K3a: per (instance, array) job cell by cell: every member's value once; for each member a
// the mismatching pairs (a, b > a) - their count into kernel kid[a]'s MISMATCH slot and the
// minimum mismatching cell into its (instance, kernel) word.  One CTA task per grid-stride
// step (pg_task_job).
__device__ __forceinline__ bool pg_pair(const PgCmp& c, u32 a, u32 b, u32 i) {
    return ((c.pair_mask >> (a * PG_MAXK + b)) & 1ull) && i < c.size[a] && i < c.size[b];
}
// the members' value rows of one instance, with their sizes (registers for the cell loop)
struct PgCmpRows {
    const u32* p[PG_MAXK];
    u32 size[PG_MAXK];
    u64 mask;
    u32 nm;
};
__device__ __forceinline__ void pg_cmp_rows(const PgCmp& c, const PgRegions& R, u32 inst, PgCmpRows& w) {
    w.nm = c.nm;
    w.mask = c.pair_mask;
#pragma unroll
    for (u32 m = 0; m < PG_MAXK; m++) {
        const bool on = m < c.nm;
        w.p[m] = on ? R.r[c.region[m]] + c.off[m] + (u64)inst * c.stride[m] : nullptr;
        w.size[m] = on ? c.size[m] : 0u;
    }
}
// one cell i: the members' values, then for each member a the mismatching pairs (a, b > a)
// (NM: members of the job - specialised, so a 2-kernel check does one pair, not 28)
template <u32 NM>
__device__ __forceinline__ void pg_cmp_vals(const PgCmpRows& w, u32 i, const u32 (&v)[PG_MAXK], u32 (&cnt)[PG_MAXK],
                                            u32 (&mn)[PG_MAXK]) {
#pragma unroll
    for (u32 a = 0; a + 1 < NM; a++) {
        u32 k = 0;
#pragma unroll
        for (u32 b = a + 1; b < NM; b++)
            k += (v[a] != v[b]) & (u32)((w.mask >> (a * PG_MAXK + b)) & 1ull) & (i < w.size[a]) & (i < w.size[b]);
        if (k) {
            cnt[a] += k;
            mn[a] = min(mn[a], i);
        }
    }
}
template <u32 NM>
__device__ __forceinline__ void pg_cmp_cell(const PgCmpRows& w, u32 i, u32 (&cnt)[PG_MAXK], u32 (&mn)[PG_MAXK]) {
    u32 v[PG_MAXK];
#pragma unroll
    for (u32 m = 0; m < NM; m++) v[m] = i < w.size[m] ? w.p[m][i] : 0u;
    pg_cmp_vals<NM>(w, i, v, cnt, mn);
}
// four consecutive cells q..q+3 (q a multiple of 4, rows 16-byte aligned): one 128-bit load
// per member, then the cells in index order
template <u32 NM>
__device__ __forceinline__ void pg_cmp_cell4(const PgCmpRows& w, u32 q, u32 (&cnt)[PG_MAXK], u32 (&mn)[PG_MAXK]) {
    uint4 v4[NM];
#pragma unroll
    for (u32 m = 0; m < NM; m++) {
        if (q + 4u <= w.size[m]) {
            v4[m] = __ldcs((const uint4*)(w.p[m] + q));
        } else {
            v4[m].x = q < w.size[m] ? w.p[m][q] : 0u;
            v4[m].y = q + 1u < w.size[m] ? w.p[m][q + 1u] : 0u;
            v4[m].z = q + 2u < w.size[m] ? w.p[m][q + 2u] : 0u;
            v4[m].w = 0u;
        }
    }
#pragma unroll
    for (u32 e = 0; e < 4u; e++) {
        u32 v[PG_MAXK];
#pragma unroll
        for (u32 m = 0; m < NM; m++) v[m] = e == 0 ? v4[m].x : e == 1 ? v4[m].y : e == 2 ? v4[m].z : v4[m].w;
        pg_cmp_vals<NM>(w, q + e, v, cnt, mn);
    }
}
// cells [lo, hi) of one instance by `lanes` threads: 128-bit streaming loads, 4 cells per
// thread per step, several steps in flight (rows are 128-byte aligned in the arenas; checked,
// the scalar loop otherwise)
template <u32 NM>
__device__ __forceinline__ void pg_cmp_range(const PgCmpRows& w, u32 lo, u32 hi, u32 lane, u32 lanes,
                                             u32 (&cnt)[PG_MAXK], u32 (&mn)[PG_MAXK]) {
    u32 al = 0;
#pragma unroll
    for (u32 m = 0; m < NM; m++) al |= (u32)(uintptr_t)w.p[m];
    if ((al & 15u) == 0u && (lo & 3u) == 0u) {
        // U steps per trip: their loads issue together (fewer for many members: registers)
        constexpr u32 U = NM <= 2 ? 4u : NM <= 4 ? 2u : 1u;
        const u32 st = 4u * lanes;
        u32 q = lo + 4u * lane;
        for (; q + (U - 1u) * st + 4u <= hi; q += U * st) {
#pragma unroll
            for (u32 u = 0; u < U; u++) pg_cmp_cell4<NM>(w, q + u * st, cnt, mn);
        }
        for (; q < hi; q += st) {
            if (q + 4u <= hi) pg_cmp_cell4<NM>(w, q, cnt, mn);
            else
                for (u32 i = q; i < hi; i++) pg_cmp_cell<NM>(w, i, cnt, mn);
        }
    } else {
        for (u32 i = lo + lane; i < hi; i += lanes) pg_cmp_cell<NM>(w, i, cnt, mn);
    }
}
template <u32 NMX>
__device__ __forceinline__ void pg_cmp_any(const PgCmpRows& w, u32 nm, u32 lo, u32 hi, u32 lane, u32 lanes,
                                           u32 (&cnt)[PG_MAXK], u32 (&mn)[PG_MAXK]) {
    if (NMX <= 2u) {   // (pairs: the kernel instance of the 2-member checks)
        pg_cmp_range<2>(w, lo, hi, lane, lanes, cnt, mn);
        return;
    }
    switch (nm) {
        case 0: case 1: case 2: pg_cmp_range<2>(w, lo, hi, lane, lanes, cnt, mn); break;
        case 3: pg_cmp_range<3>(w, lo, hi, lane, lanes, cnt, mn); break;
        case 4: pg_cmp_range<4>(w, lo, hi, lane, lanes, cnt, mn); break;
        case 5: pg_cmp_range<5>(w, lo, hi, lane, lanes, cnt, mn); break;
        case 6: pg_cmp_range<6>(w, lo, hi, lane, lanes, cnt, mn); break;
        case 7: pg_cmp_range<7>(w, lo, hi, lane, lanes, cnt, mn); break;
        default: pg_cmp_range<PG_MAXK>(w, lo, hi, lane, lanes, cnt, mn); break;
    }
}
// NMX: the most members of any job of the launch (2: pairs - 4 CTAs per SM within the
// register budget; PG_MAXK: N-kernel checks)
template <u32 NMX>
__global__ void __launch_bounds__(256, NMX <= 2 ? 4 : 2) pg_compare(const PgCmp* __restrict__ jobs, u32 n_jobs, u32 n_tasks,
                                                  const PgRegions R, PgSlot* slots, u64* mm_key) {
    __shared__ u32 s_cnt[PG_MAXK], s_min[PG_MAXK];
    __shared__ u32 s_job;
    if (threadIdx.x == 0) s_job = 0u;
    for (u32 task = blockIdx.x; task < n_tasks; task += gridDim.x) {
        const PgCmp& c = jobs[pg_task_job(jobs, n_jobs, 0u, task, &s_job)];
        const u32 lt = task - c.task0;
        u32 cnt[PG_MAXK], mn[PG_MAXK];
#pragma unroll
        for (u32 m = 0; m < PG_MAXK; m++) { cnt[m] = 0u; mn[m] = PG_NEVER; }
        if (c.n <= PG_FILL_SMALL) {   // a warp per instance
            const u32 inst = lt * 8u + (threadIdx.x >> 5), lane = threadIdx.x & 31u;
            if (inst >= c.n_inst) continue;
            PgCmpRows w;
            pg_cmp_rows(c, R, inst, w);
            pg_cmp_any<NMX>(w, c.nm, 0u, c.n, lane, 32u, cnt, mn);
#pragma unroll
            for (u32 a = 0; a + 1 < PG_MAXK; a++) {
                if (a + 1 >= c.nm) break;
                const u32 t = __reduce_add_sync(0xffffffffu, cnt[a]);
                const u32 x = __reduce_min_sync(0xffffffffu, mn[a]);
                if (lane == 0 && t) {
                    atomicAdd(&slots[c.slot0 + (u64)inst * c.slot_step + (u64)c.kid[a] * PG_NK].count, (u64)t);
                    atomicMin(&mm_key[c.mm0 + (u64)inst * c.mm_step + c.kid[a]], ((u64)c.gid << 32) | x);
                }
            }
            continue;
        }
        const u32 nch = (c.n + PG_FILL_CHUNK - 1u) / PG_FILL_CHUNK;
        const u32 inst = lt / nch, w0 = (lt - inst * nch) * PG_FILL_CHUNK, w1 = min(c.n, w0 + PG_FILL_CHUNK);
        if (threadIdx.x < PG_MAXK) { s_cnt[threadIdx.x] = 0; s_min[threadIdx.x] = PG_NEVER; }
        __syncthreads();
        PgCmpRows w;
        pg_cmp_rows(c, R, inst, w);
        pg_cmp_any<NMX>(w, c.nm, w0, w1, threadIdx.x, blockDim.x, cnt, mn);
#pragma unroll
        for (u32 a = 0; a + 1 < PG_MAXK; a++) {
            if (a + 1 >= c.nm) break;
            const u32 t = __reduce_add_sync(0xffffffffu, cnt[a]);
            const u32 x = __reduce_min_sync(0xffffffffu, mn[a]);
            if ((threadIdx.x & 31) == 0 && t) { atomicAdd(&s_cnt[a], t); atomicMin(&s_min[a], x); }
        }
        __syncthreads();
        if (threadIdx.x + 1 < c.nm && s_cnt[threadIdx.x]) {
            const u32 a = threadIdx.x;
            atomicAdd(&slots[c.slot0 + (u64)inst * c.slot_step + (u64)c.kid[a] * PG_NK].count, (u64)s_cnt[a]);
            atomicMin(&mm_key[c.mm0 + (u64)inst * c.mm_step + c.kid[a]], ((u64)c.gid << 32) | s_min[a]);
        }
        __syncthreads();
    }
}

__device__ __forceinline__ u32 pg_cmp_val(const PgCmp& c, const PgRegions& R, u32 m, u32 inst, u32 i) {
    return R.r[c.region[m]][c.off[m] + (u64)inst * c.stride[m] + i];
}
__device__ __forceinline__ u32 pg_cmp_lw(const PgCmp& c, const PgRegions& R, u32 m, u32 inst, u32 i) {
    const u32 ig = c.lwg[m] > 1u ? inst - inst % c.lwg[m] : inst;
    return ((c.lw_flags >> m) & 1u) ? R.r[c.region[m]][c.lw[m] + (u64)ig * c.stride[m] + i] - 1u : PG_NEVER;
}
__device__ __forceinline__ u32 pg_cmp_site(const PgCmp& c, u32 b) { return c.nmode ? c.kid[b] : PG_NEVER; }

// K3b: for each member a whose kernel's minimum mismatching cell lies in this job's array,
// the minimum (tid_b, site) over the pairs (a, b) that differ there - the remaining fields
// of the X16 minimum event.
__global__ void __launch_bounds__(128) pg_compare_pick(const PgCmp* __restrict__ jobs, const PgRegions R,
                                                       const u64* mm_key, u64* mm2) {
    const PgCmp& c = jobs[blockIdx.y];
    const u32 inst = blockIdx.x * blockDim.x + threadIdx.x;
    if (inst >= c.n_inst) return;
    for (u32 a = 0; a + 1 < c.nm; a++) {
        const u64 mi = c.mm0 + (u64)inst * c.mm_step + c.kid[a];
        const u64 k = mm_key[mi];
        if (k == ~0ull || (u32)(k >> 32) != c.gid) continue;
        const u32 i = (u32)k;
        if (i >= c.size[a]) continue;
        const u32 va = pg_cmp_val(c, R, a, inst, i);
        for (u32 b = a + 1; b < c.nm; b++) {
            if (!pg_pair(c, a, b, i) || pg_cmp_val(c, R, b, inst, i) == va) continue;
            atomicMin(&mm2[mi], ((u64)pg_cmp_lw(c, R, b, inst, i) << 32) | pg_cmp_site(c, b));
        }
    }
}

// K3c: fill each failing (instance, kernel kid[a]) MISMATCH record from the pair the pick chose.
__global__ void __launch_bounds__(128) pg_compare_fill(const PgCmp* __restrict__ jobs, const PgRegions R,
                                                       PgSlot* slots, const u64* mm_key, const u64* mm2) {
    const PgCmp& c = jobs[blockIdx.y];
    const u32 inst = blockIdx.x * blockDim.x + threadIdx.x;
    if (inst >= c.n_inst) return;
    for (u32 a = 0; a + 1 < c.nm; a++) {
        const u64 mi = c.mm0 + (u64)inst * c.mm_step + c.kid[a];
        const u64 k = mm_key[mi];
        if (k == ~0ull || (u32)(k >> 32) != c.gid) continue;
        const u32 i = (u32)k;
        if (i >= c.size[a]) continue;
        const u32 va = pg_cmp_val(c, R, a, inst, i);
        for (u32 b = a + 1; b < c.nm; b++) {
            if (!pg_pair(c, a, b, i)) continue;
            const u32 vb = pg_cmp_val(c, R, b, inst, i);
            const u32 tb = pg_cmp_lw(c, R, b, inst, i);
            if (vb == va || mm2[mi] != (((u64)tb << 32) | pg_cmp_site(c, b))) continue;
            PgSlot* s = &slots[c.slot0 + (u64)inst * c.slot_step + (u64)c.kid[a] * PG_NK];
            s->f[0] = 0xFFFFu;
            s->f[1] = c.gid;
            s->f[2] = i;
            s->f[3] = pg_cmp_lw(c, R, a, inst, i);
            s->f[4] = tb;
            s->f[5] = pg_cmp_site(c, b);
            s->f[6] = va;
            s->f[7] = vb;
            s->has = 1u;
            break;
        }
    }
}

// K2b: flag every instance in which some global cell written by the kernel was
// accessed by two blocks (X4 XB) - the block-parallel pass is not exact there.
__global__ void __launch_bounds__(256) pg_xb_detect(const PgXb* __restrict__ jobs, u32 n_jobs, u32 n_tasks,
                                                    const u32* arena, u32* flags, u32* any, const u32* pref) {
    __shared__ u32 s_job;
    if (threadIdx.x == 0) s_job = 0u;
    for (u32 task = blockIdx.x; task < n_tasks; task += gridDim.x) {
        const PgXb j = jobs[pg_task_job(jobs, n_jobs, 0u, task, &s_job)];
        const u32 lt = task - j.task0;
        const u32 nb = (j.n_inst + j.istep - 1u) / j.istep;   // instances holding marks
        auto flag = [&](u32 b) {   // the group of instance b * istep
            const u32 i0 = b * j.istep, i1 = min(j.n_inst, i0 + j.istep);
            for (u32 i = i0; i < i1; i++) flags[j.inst0 + i] = 1u;
            *any = 1u;
        };
        // (launches the sequential pass takes whole: the parallel passes skipped them)
        const bool all = pref != nullptr && pref[j.launch] != 0u;
        if (j.n <= PG_FILL_SMALL) {   // a warp per instance
            const u32 b = lt * 8u + (threadIdx.x >> 5), lane = threadIdx.x & 31u;
            if (b >= nb) continue;
            if (all) {
                if (lane == 0) flag(b);
                continue;
            }
            const u64 base = (u64)b * j.istep * j.stride;
            u32 hit = 0;
            for (u32 i = lane; i < j.n; i += 32u) {
                const u32 xf = arena[j.xf + base + i], xl = arena[j.xl + base + i];
                hit |= (xl != 0u && xf != xl && arena[j.lw + base + i] != 0u);
            }
            if (__any_sync(0xffffffffu, hit) && lane == 0) flag(b);
            continue;
        }
        const u32 nch = (j.n + PG_FILL_CHUNK - 1u) / PG_FILL_CHUNK;
        const u32 b = lt / nch, w0 = (lt - b * nch) * PG_FILL_CHUNK, w1 = min(j.n, w0 + PG_FILL_CHUNK);
        if (all) {
            if (threadIdx.x == 0 && w0 == 0) flag(b);
            continue;
        }
        const u64 base = (u64)b * j.istep * j.stride;
        u32 hit = 0;
        for (u32 i = w0 + threadIdx.x; i < w1; i += blockDim.x) {
            const u32 xf = arena[j.xf + base + i], xl = arena[j.xl + base + i], lw = arena[j.lw + base + i];
            hit |= (xl != 0u) & (xf != xl) & (lw != 0u);
        }
        if (__syncthreads_or((int)hit) && threadIdx.x == 0) flag(b);
    }
}

// K3b: lock-step comparison (X25).  Per (instance, matched shared array): the smallest
// (block, round, array, cell) at which both kernels took a snapshot and the (value,
// written) pairs differ, as key = block << 34 | round << 29 | array << 24 | cell, min-reduced
// into keys[instance].  Snapshots never taken are all-ones (K1 fill).
__device__ __forceinline__ u64 pg_lock_key(const PgLock& j, u64 i) {
    const u64 cell = i % j.size, br = i / j.size;
    return ((br / j.rounds) << 34) | ((br % j.rounds) << 29) | ((u64)j.arr_slot << 24) | cell;
}
__global__ void __launch_bounds__(256) pg_lockstep_cmp(const PgLock* __restrict__ jobs, const u32* arena_s,
                                                       const u32* arena_t, u64* keys) {
    const PgLock j = jobs[blockIdx.y];
    const u64 n = (u64)j.nblocks * j.rounds * j.size;
    for (u32 inst = blockIdx.x; inst < j.n_inst; inst += gridDim.x) {
        const uint2* s = (const uint2*)(arena_s + j.src_off + (u64)inst * j.src_stride);
        const uint2* t = (const uint2*)(arena_t + j.tgt_off + (u64)inst * j.tgt_stride);
        u64 best = ~0ull;
        for (u64 i = threadIdx.x; i < n; i += blockDim.x) {   // i order = key order for one array
            const uint2 a = s[i], b = t[i];
            if ((a.x & a.y) == PG_NEVER || (b.x & b.y) == PG_NEVER) continue;   // a round one kernel lacks
            if (a.x != b.x || a.y != b.y) {
                best = pg_lock_key(j, i);
                break;
            }
        }
        for (int o = 16; o > 0; o >>= 1) {
            const u64 x = __shfl_down_sync(0xFFFFFFFFu, best, o);
            best = x < best ? x : best;
        }
        if ((threadIdx.x & 31u) == 0u && best != ~0ull) atomicMin((unsigned long long*)&keys[j.key0 + inst], best);
    }
}
// rows (10 words per instance) for the instances whose minimum lies in this job's array
__global__ void __launch_bounds__(128) pg_lockstep_fill(const PgLock* __restrict__ jobs, const u32* arena_s,
                                                        const u32* arena_t, const u64* keys, u32* rows, u32 n_local,
                                                        u32 rank, u32 world) {
    const PgLock j = jobs[blockIdx.y];
    const u32 inst = blockIdx.x * blockDim.x + threadIdx.x;
    if (inst >= j.n_inst) return;
    const u64 gi = j.key0 + inst, key = keys[gi];
    if (key == ~0ull || ((key >> 24) & 31u) != j.arr_slot) return;
    const u64 blk = key >> 34, round = (key >> 29) & 31u, cell = key & 0xFFFFFFu;
    const u64 i = (blk * j.rounds + round) * j.size + cell;
    const uint2 a = ((const uint2*)(arena_s + j.src_off + (u64)inst * j.src_stride))[i];
    const uint2 b = ((const uint2*)(arena_t + j.tgt_off + (u64)inst * j.tgt_stride))[i];
    u32* r = rows + gi * 10u;
    r[0] = (u32)(gi / n_local);
    r[1] = rank + (u32)(gi % n_local) * world;
    r[2] = (u32)blk; r[3] = (u32)round; r[4] = 0x100u + j.arr_slot; r[5] = (u32)cell;
    r[6] = a.x; r[7] = b.x; r[8] = a.y; r[9] = b.y;
}

// K2b': list the sequential-pass items whose seed group has a flagged instance.
__global__ void __launch_bounds__(256) pg_seq_select(const PgWork* __restrict__ items, u32 n_items,
                                                     const u32* flags, u32* list, u32* count) {
    const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_items) return;
    const PgWork w = items[i];
    u32 f = 0;
    for (u32 s = 0; s < w.nseeds; s++) f |= flags[w.inst0 + s];
    if (f) list[atomicAdd(count, 1u)] = i;
}

// K2c: fold the per-item site statistics of the block-parallel pass into the
// per-launch table, skipping seed groups that the sequential pass re-runs.
__global__ void __launch_bounds__(128) pg_stats_reduce(const PgWork* __restrict__ items, const u64* item_stats,
                                                       u32* flags, u64* launch_stats, u32 max_sites) {
    const PgWork w = items[blockIdx.x];
    __shared__ u32 s_skip;
    if (threadIdx.x == 0) {
        u32 f = 0;
        for (u32 i = 0; i < w.nseeds; i++) f |= flags[w.inst0 + i];
        s_skip = f;
    }
    __syncthreads();
    if (s_skip) {
        // the sequential pass recomputes this item's statistics: make it re-run every seed of
        // the item (a multi-seed item holds several whole one-seed sequential items)
        for (u32 i = threadIdx.x; i < w.nseeds; i += blockDim.x) flags[w.inst0 + i] = 1u;
        return;
    }
    const u64* src = item_stats + (u64)w.item * max_sites * 8u;
    u64* dst = launch_stats + (u64)w.launch * max_sites * 8u;
    for (u32 i = threadIdx.x; i < max_sites * 8u; i += blockDim.x) {
        const u64 v = src[i];
        if (!v) continue;
        const u32 c = i & 7u;
        if (c == 0) dst[i] = v;
        else if (c == 3) atomicMax(&dst[i], v);
        else atomicAdd(&dst[i], v);
    }
}

__global__ void pg_reset_counters(long long* first_key, long long* counts) {
    const u32 i = threadIdx.x;
    if (i < 11) first_key[i] = 0x7FFFFFFFFFFFFFFFll;
    if (i < 16) counts[i] = 0;
}

// K5: merge the counters of several checks (rows of first keys int64[11] and counts
// int64[16]): MIN of the keys, SUM of the counts - the same reduction H9 applies across ranks.
__global__ void pg_merge_counters(const long long* keys, const long long* counts, u32 n, long long* out_keys,
                                  long long* out_counts) {
    const u32 i = threadIdx.x;
    if (i < 11) {
        long long m = 0x7FFFFFFFFFFFFFFFll;
        for (u32 r = 0; r < n; r++) m = min(m, keys[(u64)r * 11u + i]);
        out_keys[i] = m;
    }
    if (i < 16) {
        long long s = 0;
        for (u32 r = 0; r < n; r++) s += counts[(u64)r * 16u + i];
        out_counts[i] = s;
    }
}

__device__ __forceinline__ bool kind_failing(u32 kind, u32 banks_mode) {
    return kind <= PGK_MISMATCH || kind == PGK_LIMIT || (banks_mode && (kind == PGK_BANK || kind == PGK_UNCOAL));
}

// K4a: per instance (launch, local seed m): count non-empty slots, fold counts
// and keys into the summary (X16/X17).
__global__ void __launch_bounds__(256) pg_summarize(const PgSlot* __restrict__ slots, u32 n_inst, u32 n_local,
                                                    u32 rank, u32 world, u32 banks_mode, u32 nks, u32 l0, u32 s0,
                                                    u32* inst_nrec, long long* first_key, long long* counts) {
    const u32 inst = blockIdx.x * blockDim.x + threadIdx.x;
    if (inst >= n_inst) return;
    const u32 li = l0 + inst / n_local, m = inst % n_local;
    const u32 sj = s0 + rank + m * world;
    u32 n = 0, failing = 0;
    for (u32 k = 0; k < nks; k++) {
        for (u32 kind = 0; kind < PG_NK; kind++) {
            const PgSlot& s = slots[((u64)inst * nks + k) * PG_NK + kind];
            if (s.count == 0 || !s.has) continue;
            n++;
            const long long key = (long long)(((u64)li << 45) | ((u64)sj << 24) | ((u64)k << 20) |
                                              ((u64)kind << 16) | (u64)(s.f[0] & 0xFFFFu));
            atomicAdd((unsigned long long*)&counts[1 + kind], (unsigned long long)s.count);
            atomicMin(&first_key[1 + kind], key);
            if (kind_failing(kind, banks_mode)) {
                failing = 1;
                atomicMin(&first_key[0], key);
            }
        }
    }
    inst_nrec[inst] = n;
    if (n) atomicAdd((unsigned long long*)&counts[11], (unsigned long long)n);
    if (failing) atomicAdd((unsigned long long*)&counts[12], 1ull);
}

// K4b: exclusive scan of per-instance record counts (one CTA; chunked).
__global__ void __launch_bounds__(1024) pg_scan(const u32* in, u64* out, u32 n) {
    __shared__ u64 warp_sums[32];
    __shared__ u64 carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (u32 base = 0; base < n; base += 1024) {
        const u32 i = base + threadIdx.x;
        u64 v = i < n ? in[i] : 0;
        const u32 lane = threadIdx.x & 31, w = threadIdx.x >> 5;
        u64 x = v;
        for (int o = 1; o < 32; o <<= 1) {
            u64 y = __shfl_up_sync(0xffffffffu, x, o);
            if (lane >= (u32)o) x += y;
        }
        if (lane == 31) warp_sums[w] = x;
        __syncthreads();
        if (w == 0) {
            u64 s = warp_sums[lane];
            for (int o = 1; o < 32; o <<= 1) {
                u64 y = __shfl_up_sync(0xffffffffu, s, o);
                if (lane >= (u32)o) s += y;
            }
            warp_sums[lane] = s;
        }
        __syncthreads();
        const u64 incl = x + (w ? warp_sums[w - 1] : 0) + carry;
        if (i < n) out[i] = incl - v;
        __syncthreads();
        if (threadIdx.x == 1023) carry = incl;
        __syncthreads();
    }
}

struct PgCexDev {
    u64 key, count;
    u32 kind, launch, seed_idx, kernel, round, site, array, addr, tid_a, tid_b, val_a, val_b;
};

// K4c: write each instance's records at its scanned offset (slot order = key order).
// The run's record count (its own records, before any cross-rank reduction of the counters)
// goes to *total.
__global__ void __launch_bounds__(256) pg_compact(const PgSlot* __restrict__ slots, u32 n_inst, u32 n_local,
                                                  u32 rank, u32 world, u32 nks, u32 l0, u32 s0, const u32* inst_nrec,
                                                  const u64* offsets, PgCexDev* out, u64 cap, u64* total) {
    const u32 inst = blockIdx.x * blockDim.x + threadIdx.x;
    if (inst == 0) *total = offsets[n_inst - 1] + inst_nrec[n_inst - 1];
    if (inst >= n_inst) return;
    const u32 li = l0 + inst / n_local, m = inst % n_local;
    const u32 sj = s0 + rank + m * world;
    u64 o = offsets[inst];
    for (u32 k = 0; k < nks; k++) {
        for (u32 kind = 0; kind < PG_NK; kind++) {
            const PgSlot& s = slots[((u64)inst * nks + k) * PG_NK + kind];
            if (s.count == 0 || !s.has) continue;
            if (o < cap) {
                PgCexDev r;
                r.key = ((u64)li << 45) | ((u64)sj << 24) | ((u64)k << 20) | ((u64)kind << 16) | (u64)(s.f[0] & 0xFFFFu);
                r.count = s.count;
                r.kind = kind;
                r.launch = li;
                r.seed_idx = sj;
                r.kernel = k;
                r.round = s.f[0];
                r.array = s.f[1];
                r.addr = s.f[2];
                r.tid_a = s.f[3];
                r.tid_b = s.f[4];
                r.site = s.f[5];
                r.val_a = s.f[6];
                r.val_b = s.f[7];
                out[o] = r;
            }
            o++;
        }
    }
}

// Before the exact re-run of flagged instances: clear their record slots (this kernel)
// and their instance counts.
__global__ void __launch_bounds__(256) pg_reset_flagged(const u32* flags, u32 n_inst, const u64* inst_slot0,
                                                        u32 kernel, PgSlot* slots, u64* inst_cnt,
                                                        u32* flag_count) {
    const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
    if (!flags[n_inst]) return;   // (the batch's any-flagged word)
    const u32 f = i < n_inst && flags[i] != 0u;
    if (flag_count) {   // flagged instances of the check (the planner's choice of main pass)
        const u32 c = __popc(__ballot_sync(0xffffffffu, f));
        if ((threadIdx.x & 31u) == 0u && c) atomicAdd(flag_count, c);
    }
    if (!f) return;
    inst_cnt[i] = 0ull;
    PgSlot* s = slots + inst_slot0[i] + (u64)kernel * PG_NK;
    for (u32 k = 0; k < PG_NK; k++) {
        s[k].count = 0ull;
        s[k].lock = 0u;
        s[k].has = 0u;
        s[k].pkey = 0ull;
    }
}

// Sequential preference (PgParams::seq_pref): the instances whose sequential run found an XB
// race (flag word 2), counted per launch (launch = record slot / (n_local x slots per seed)).
__global__ void __launch_bounds__(256) pg_xb_tally(const u32* flags, u32 n_inst, const u64* inst_slot0, u64 div,
                                                   u32* counts, u32* total) {
    const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
    if (!flags[n_inst]) return;
    const u32 x = i < n_inst && flags[i] == 2u;
    if (x && counts) atomicAdd(&counts[inst_slot0[i] / div], 1u);
    const u32 c = __popc(__ballot_sync(0xffffffffu, x));   // (the host's count: any XB at all)
    if ((threadIdx.x & 31u) == 0u && c) atomicAdd(total, c);
}
// After the check: a launch goes straight to the sequential pass next time iff at least half
// of its instances here raced between blocks (re-decided every check); counts reset.
__global__ void __launch_bounds__(256) pg_seq_pref_update(u32* counts, u32* pref, u32 n, u32 n_local) {
    const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    pref[i] = 2u * counts[i] >= n_local && counts[i] != 0u ? 1u : 0u;
    counts[i] = 0u;
}

// X19: the batch's per-instance counts into the run's instance counter.
__global__ void __launch_bounds__(1024) pg_count_reduce(const u64* inst_cnt, u32 n, unsigned long long* counts) {
    u64 x = 0;
    for (u32 i = threadIdx.x; i < n; i += blockDim.x) x += inst_cnt[i];
    for (int o = 16; o > 0; o >>= 1) x += __shfl_down_sync(0xffffffffu, x, o);
    __shared__ u64 part[32];
    if ((threadIdx.x & 31u) == 0u) part[threadIdx.x >> 5] = x;
    __syncthreads();
    if (threadIdx.x == 0) {
        u64 t = 0;
        for (u32 w = 0; w < (blockDim.x + 31u) / 32u; w++) t += part[w];
        atomicAdd(counts, t);
    }
}

// Condition of a captured re-run block (a conditional IF node of the check graph): run the
// block only if some instance of the batch was flagged.
__global__ void pg_set_cond(cudaGraphConditionalHandle h, const u32* flag) {
    cudaGraphSetConditional(h, *(volatile const u32*)flag != 0u ? 1u : 0u);
}

// ------------------------------------------------------------------ INT32 peak microbenchmark
// Measurement only (the roofline denominator of K2): 8 independent
// chains per thread of LOP3 (alu pipe, mode 0), IMAD (fma pipe, mode 1) or both
// alternating (mode 2), 16 x 8 = 128 integer ops per loop trip.  inline PTX keeps ptxas
// from folding the chains; the result is stored only under a condition it cannot decide.
template <int MODE>
__global__ void __launch_bounds__(256) pg_int_peak(u32 iters, u32* sink) {
    u32 a[8];
    const u32 b = threadIdx.x * 0x9E3779B9u + blockIdx.x, c = (u32)clock() | 1u;
#pragma unroll
    for (int j = 0; j < 8; j++) a[j] = b + (u32)j * 0x85EBCA6Bu;
    for (u32 i = 0; i < iters; i++) {
#pragma unroll
        for (int r = 0; r < 16; r++) {
#pragma unroll
            for (int j = 0; j < 8; j++) {
                if (MODE == 0 || (MODE == 2 && (j & 1)))
                    asm volatile("lop3.b32 %0, %0, %1, %2, 0x6A;" : "+r"(a[j]) : "r"(b), "r"(c));
                else
                    asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(a[j]) : "r"(c), "r"(b));
            }
        }
    }
    u32 x = 0;
#pragma unroll
    for (int j = 0; j < 8; j++) x ^= a[j];
    if (x == 0x1234567u && b == c) sink[threadIdx.x] = x;
}

}  // namespace

// ------------------------------------------------------------------ host wrappers (C++ linkage, used by api.cpp)
namespace pgk {

// SMs of the current device (queried once per device): grids of the CTA-task kernels stride
// over their tasks with <= 16 CTAs per SM
u32 sm_count() {
    static int cache[64] = {0};
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 148u;
    if (!cache[dev]) {
        int n = 0;
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        cache[dev] = n > 0 ? n : 148;
    }
    return (u32)cache[dev];
}
u32 task_grid(u32 n_tasks) { return n_tasks < sm_count() * 16u ? n_tasks : sm_count() * 16u; }


cudaError_t gen_inputs(const PgFill* jobs, u32 n_jobs, u32 task_base, u32 n_tasks, const PgRegions& R,
                       u64 seed_base, u32 mode, u32 range, u32 mask, cudaStream_t st, const u32* flags,
                       const u32* any) {
    if (!n_jobs || !n_tasks) return cudaSuccess;
    const u32 grid = task_grid(n_tasks);
    pg_gen_inputs<<<grid, 256, 0, st>>>(jobs, n_jobs, task_base, n_tasks, R, seed_base, mode, range, mask, flags,
                                        any);
    return cudaGetLastError();
}

cudaError_t reset_flagged(const u32* flags, u32 n_inst, const u64* inst_slot0, u32 kernel, PgSlot* slots,
                          u64* inst_cnt, u32* flag_count, cudaStream_t st) {
    if (!n_inst) return cudaSuccess;
    pg_reset_flagged<<<(n_inst + 255) / 256, 256, 0, st>>>(flags, n_inst, inst_slot0, kernel, slots, inst_cnt,
                                                           flag_count);
    return cudaGetLastError();
}

cudaError_t xb_tally(const u32* flags, u32 n_inst, const u64* inst_slot0, u64 div, u32* counts, u32* total,
                     cudaStream_t st) {
    if (!n_inst) return cudaSuccess;
    pg_xb_tally<<<(n_inst + 255) / 256, 256, 0, st>>>(flags, n_inst, inst_slot0, div, counts, total);
    return cudaGetLastError();
}

cudaError_t seq_pref_update(u32* counts, u32* pref, u32 n, u32 n_local, cudaStream_t st) {
    if (!n) return cudaSuccess;
    pg_seq_pref_update<<<(n + 255) / 256, 256, 0, st>>>(counts, pref, n, n_local);
    return cudaGetLastError();
}

cudaError_t count_reduce(const u64* inst_cnt, u32 n, long long* counts, cudaStream_t st) {
    if (!n) return cudaSuccess;
    pg_count_reduce<<<1, 1024, 0, st>>>(inst_cnt, n, (unsigned long long*)counts);
    return cudaGetLastError();
}

cudaError_t compare(const PgCmp* jobs, u32 n_jobs, u32 n_tasks, u32 max_nm, u32 max_inst, const PgRegions& R,
                    PgSlot* slots, u64* mm_key, u64* mm2, cudaStream_t st) {
    if (!n_jobs) return cudaSuccess;
    if (max_nm <= 2u) pg_compare<2><<<task_grid(n_tasks), 256, 0, st>>>(jobs, n_jobs, n_tasks, R, slots, mm_key);
    else pg_compare<PG_MAXK><<<task_grid(n_tasks), 256, 0, st>>>(jobs, n_jobs, n_tasks, R, slots, mm_key);
    for (u32 j0 = 0; j0 < n_jobs; j0 += 65535u) {
        const u32 nj = n_jobs - j0 < 65535u ? n_jobs - j0 : 65535u;
        dim3 g2((max_inst + 127) / 128, nj);
        pg_compare_pick<<<g2, 128, 0, st>>>(jobs + j0, R, mm_key, mm2);
    }
    for (u32 j0 = 0; j0 < n_jobs; j0 += 65535u) {
        const u32 nj = n_jobs - j0 < 65535u ? n_jobs - j0 : 65535u;
        dim3 g2((max_inst + 127) / 128, nj);
        pg_compare_fill<<<g2, 128, 0, st>>>(jobs + j0, R, slots, mm_key, mm2);
    }
    return cudaGetLastError();
}

cudaError_t lockstep(const PgLock* jobs, u32 n_jobs, u32 max_inst, const u32* arena_s, const u32* arena_t, u64* keys,
                     u32* rows, u32 n_local, u32 rank, u32 world, cudaStream_t st) {
    for (u32 j0 = 0; j0 < n_jobs; j0 += 65535u) {
        const u32 nj = n_jobs - j0 < 65535u ? n_jobs - j0 : 65535u;
        dim3 grid(max_inst < 1024u ? max_inst : 1024u, nj);
        pg_lockstep_cmp<<<grid, 256, 0, st>>>(jobs + j0, arena_s, arena_t, keys);
        dim3 g2((max_inst + 127) / 128, nj);
        pg_lockstep_fill<<<g2, 128, 0, st>>>(jobs + j0, arena_s, arena_t, keys, rows, n_local, rank, world);
    }
    return cudaGetLastError();
}

cudaError_t xb_detect(const PgXb* jobs, u32 n_jobs, u32 n_tasks, const u32* arena, u32* flags, u32* any,
                      const u32* pref, cudaStream_t st) {
    if (!n_jobs || !n_tasks) return cudaSuccess;
    pg_xb_detect<<<task_grid(n_tasks), 256, 0, st>>>(jobs, n_jobs, n_tasks, arena, flags, any, pref);
    return cudaGetLastError();
}

cudaError_t seq_select(const PgWork* items, u32 n_items, const u32* flags, u32* list, u32* count, cudaStream_t st) {
    if (!n_items) return cudaSuccess;
    pg_seq_select<<<(n_items + 255) / 256, 256, 0, st>>>(items, n_items, flags, list, count);
    return cudaGetLastError();
}

cudaError_t stats_reduce(const PgWork* items, u32 n_items, const u64* item_stats, u32* flags, u64* launch_stats,
                         u32 max_sites, cudaStream_t st) {
    if (!n_items) return cudaSuccess;
    pg_stats_reduce<<<n_items, 128, 0, st>>>(items, item_stats, flags, launch_stats, max_sites);
    return cudaGetLastError();
}

cudaError_t merge_counters(const long long* keys, const long long* counts, u32 n, long long* out_keys,
                           long long* out_counts, cudaStream_t st) {
    pg_merge_counters<<<1, 32, 0, st>>>(keys, counts, n, out_keys, out_counts);
    return cudaGetLastError();
}

cudaError_t reset_counters(long long* first_key, long long* counts, cudaStream_t st) {
    pg_reset_counters<<<1, 32, 0, st>>>(first_key, counts);
    return cudaGetLastError();
}

cudaError_t summarize_scan(const PgSlot* slots, u32 n_inst, u32 n_local, u32 rank, u32 world, u32 banks_mode,
                           u32 nks, u32 l0, u32 s0, u32* inst_nrec, u64* offsets, long long* first_key,
                           long long* counts, cudaStream_t st) {
    if (!n_inst) return cudaSuccess;
    pg_summarize<<<(n_inst + 255) / 256, 256, 0, st>>>(slots, n_inst, n_local, rank, world, banks_mode, nks, l0, s0,
                                                       inst_nrec, first_key, counts);
    pg_scan<<<1, 1024, 0, st>>>(inst_nrec, offsets, n_inst);
    return cudaGetLastError();
}

cudaError_t compact(const PgSlot* slots, u32 n_inst, u32 n_local, u32 rank, u32 world, u32 nks, u32 l0, u32 s0,
                    const u32* inst_nrec, const u64* offsets, void* out, u64 cap, u64* total, cudaStream_t st) {
    if (!n_inst) return cudaSuccess;
    pg_compact<<<(n_inst + 255) / 256, 256, 0, st>>>(slots, n_inst, n_local, rank, world, nks, l0, s0, inst_nrec,
                                                     offsets, (PgCexDev*)out, cap, total);
    return cudaGetLastError();
}

cudaError_t set_cond(cudaGraphConditionalHandle h, const u32* flag, cudaStream_t st) {
    pg_set_cond<<<1, 1, 0, st>>>(h, flag);
    return cudaGetLastError();
}

cudaError_t int_peak(int mode, u32 blocks, u32 iters, u32* sink, cudaStream_t st) {
    if (mode == 0) pg_int_peak<0><<<blocks, 256, 0, st>>>(iters, sink);
    else if (mode == 1) pg_int_peak<1><<<blocks, 256, 0, st>>>(iters, sink);
    else pg_int_peak<2><<<blocks, 256, 0, st>>>(iters, sink);
    return cudaGetLastError();
}

}  // namespace pgk
