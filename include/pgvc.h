/*
 * pgvc.h — C ABI of libpgvc.so: bounded, exhaustive instantiation of PUGpara's
 * parameterized verification conditions on a B200.
 *
 * Paper: G. Li, G. Gopalakrishnan, "Parameterized Verification of GPU Kernel
 * Programs" (/root/reference/PAPER.md, cited Lnnn).  Semantics readings X1-X21
 * are in DESIGN.md §2.
 *
 * Conventions
 *   - Every function returns a PG_* status (0 = success); no C++ exception
 *     crosses this boundary.  pg_last_error() returns a thread-local message
 *     ("line:col: ..." for parse/type errors), valid until the next call on the
 *     same thread.
 *   - Handles (pg_ir, pg_run) are owned by the caller and freed with
 *     pg_ir_free / pg_run_free.  A pg_run owns its device and host buffers.
 *   - Pointers in pg_space are borrowed for the duration of the call, except
 *     d_first_key / d_counts / cuda_stream, which are borrowed (owned by the
 *     caller, e.g. torch) until pg_collect_cex returns.
 *   - pg_check_* only ENQUEUE work on cuda_stream; pg_collect_cex synchronises
 *     that stream.  No collective is issued by the library: the caller may
 *     all_reduce d_first_key (MIN) and d_counts (SUM) between pg_check_* and
 *     pg_collect_cex (H9).
 *   - There is no CPU fallback: without a usable CUDA device every check
 *     returns PG_E_CUDA.
 */
#ifndef PGVC_H
#define PGVC_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct pg_ir pg_ir;    /* one loaded kernel: parsed, checked, code-generated; immutable */
typedef struct pg_run pg_run;  /* result set of one check */

enum {
    PG_OK = 0,
    PG_E_ARG = -1,    /* bad argument */
    PG_E_PARSE = -2,  /* syntax error in the kernel text (line:col in pg_last_error) */
    PG_E_TYPE = -3,   /* semantic error: undeclared name, sync under thread-dependent control (X18), ... */
    PG_E_LIMIT = -4,  /* static or launch limit exceeded (arrays > 2^24 words, > 4096 threads/block, ...) */
    PG_E_CUDA = -5,   /* CUDA driver / runtime / NVRTC failure, or no device */
    PG_E_OOM = -6,    /* device allocation failed */
    PG_E_STATE = -7   /* call out of order (e.g. collect on a run that was never checked) */
};

enum { PG_IN_RAND32 = 0, PG_IN_BITS01 = 1, PG_IN_RANGE = 2 };                 /* X8 */
enum { PG_CHK_EQUIV = 1, PG_CHK_RACE = 2, PG_CHK_OOB = 4, PG_CHK_BANK = 8, PG_CHK_COALESCE = 16,
       PG_CHK_DATAFLOW = 32, /* record the writer of every read (H5); evaluates blocks in bid order */
       PG_CHK_LOCKSTEP = 64, /* pg_check_equiv: compare the kernels' shared state round by round */
       PG_CHK_VCLITERAL = 256, /* with PG_CHK_DATAFLOW (implied): blocks of <= 64 threads; each read's writer
                                  is also found literally on the device - every thread s of every earlier
                                  round tested for "s wrote the cell" (the instantiated p(s) /\ a = e(s),
                                  L521-L522, L709-L712) - and compared with the owner-stamp writer
                                  (pg_collect_vcliteral) */
       PG_CHK_OPCOUNT = 128  /* measurement: count the IR integer operations the kernels execute (each
                                unary / binary / logical / select / min / max node and two per extra array
                                dimension, under the thread's predicate) into d_counts[13]; exact
                                single-seed passes */ };
enum { PG_LOCK_ROUNDS = 32 };   /* rounds of every block the lock-step comparison covers */
enum { PG_BANKS_32 = 0, PG_BANKS_16_HALFWARP = 1 };                             /* X9 */
enum {                                                                          /* X17 */
    PG_CEX_BARRIER_DIV = 0, PG_CEX_OOB = 1, PG_CEX_RACE_WW = 2, PG_CEX_RACE_RW = 3, PG_CEX_RACE_XB = 4,
    PG_CEX_MISMATCH = 5, PG_CEX_BANK = 6, PG_CEX_UNCOALESCED = 7, PG_CEX_UNINIT = 8, PG_CEX_LIMIT = 9,
    PG_N_KINDS = 10
};

/* One value of the paper's parameter n (L110-L116): grid and block shape plus
 * the kernel's scalar parameters in declaration order. */
typedef struct {
    uint32_t gdim[3], bdim[3];
    int32_t scalar[8];
    uint32_t n_scalar;
} pg_launch;

/* The bounded parameter space of one check (H1).  launch_src[i] and
 * launch_tgt[i] describe the same point n for the two kernels (the target may
 * use another block shape, e.g. reduce3 uses bdim = B/2); index order is the
 * witness order (X16).  Seeds seed_base + j for j in [0, n_seeds); this call
 * covers the shard j = rank, rank + world, ... */
typedef struct {
    const pg_launch *launch_src, *launch_tgt;  /* launch_tgt may be NULL (= launch_src) */
    uint32_t n_launch;                         /* < 2^18 */
    uint64_t seed_base;
    uint32_t n_seeds;                          /* < 2^21 */
    uint32_t input_mode, input_range;          /* PG_IN_*, k for PG_IN_RANGE */
    uint32_t bits;                             /* arithmetic width w (X2): 1..32, default 32 */
    uint32_t checks, bank_model, max_cex;      /* PG_CHK_* mask; PG_BANKS_*; max records kept */
    int32_t rank, world;                       /* shard of (launch, seed) instances */
    void *cuda_stream;                         /* borrowed cudaStream_t (0 = legacy default stream) */
    int64_t *d_first_key;                      /* borrowed device int64[11]: [0] min failing key, [1+k] min key of kind k; INT64_MAX = none */
    int64_t *d_counts;                         /* borrowed device int64[16]: [0] instances (X19), [1+k] events of kind k,
                                                  [11] records, [12] failing (launch, seed) instances,
                                                  [13] IR operations executed (PG_CHK_OPCOUNT only) */
    uint32_t key_launch0, key_seed0;           /* added to the launch index and the seed index of every key and
                                                  record: a sub-space (some launches x a seed range, e.g. one item
                                                  of a greedy (launch, seed) assignment, §8(e)) reports the keys of
                                                  the whole space, so sub-space results merge like rank shards.
                                                  0 for a whole space */
} pg_space;

/* One counterexample record (X16): the minimum event of its (launch, seed,
 * kernel, kind) slot, and the slot's event count.  tid_a/tid_b are global
 * linear thread ids (XB: block ids).  key = launch (19 bits) | seed_idx (21) |
 * kernel (4) | kind (4) | round (16; 0xFFFF for MISMATCH / XB). */
typedef struct {
    uint64_t key, count;
    uint32_t kind, launch, seed_idx, kernel, round, site, array, addr, tid_a, tid_b, val_a, val_b;
} pg_cex;

typedef struct {
    uint64_t instances;        /* X19 */
    uint64_t n_fail;           /* failing (launch, seed) instances */
    uint64_t n_records;
    int64_t first_key;         /* min failing key (INT64_MAX: none) */
    uint32_t first_launch;     /* launch index of first_key (0xFFFFFFFF: none) = first-witness n */
    uint32_t first_seed_idx;
    uint64_t per_kind[PG_N_KINDS];
    int64_t first_key_kind[PG_N_KINDS];
    uint64_t ir_ops;           /* d_counts[13]: IR operations executed (PG_CHK_OPCOUNT runs) */
} pg_summary;

/* Parse, check and code-generate one kernel (the IR of DESIGN.md §4; the
 * paper's C subset, L122-L171).  `text` need not be NUL-terminated.
 * Errors: PG_E_PARSE / PG_E_TYPE with line:col, PG_E_LIMIT. */
int pg_load_ir(const char *text, size_t len, pg_ir **out);

/* Comparative assertion (L438-L444, L652-L657): both kernels on every launch
 * and seed of the space, same initial global arrays (X7), compare every array
 * that is out/inout in either kernel; plus the checks selected in sp->checks
 * (RACE: WW/RW/XB; OOB: out-of-bounds and uninitialised reads; BANK/COALESCE
 * report-only).  Enqueues on sp->cuda_stream. */
int pg_check_equiv(const pg_ir *src, const pg_ir *tgt, const pg_space *sp, pg_run **out);

/* N-kernel comparative assertion (SURVEY.md §8(d) C2 design: reduce0..6 pairwise): nk
 * kernels (2..8), kernel k with launch list launches[k] (n_launch points each, the same
 * parameter n in the same order; NULL entry or NULL array = sp->launch_src), each evaluated
 * ONCE per (launch, seed), then every pair i < j compared on every global array that is
 * out/inout in either (matched by name).  A mismatch of the pair (i, j) is an event of kernel
 * i's MISMATCH slot with site = j (the slot's record is the minimum over j, X16; its count
 * sums the mismatching cells of every pair).  Races / OOB / LIMIT per kernel as in
 * pg_check_equiv.  BANK / COALESCE / LOCKSTEP are PG_E_ARG (pair checks). */
int pg_check_equiv_n(const pg_ir *const *ks, uint32_t nk, const pg_launch *const *launches, const pg_space *sp,
                     pg_run **out);

/* Multi-kernel sequences (GKLEE's multi-kernel programs L62-L63):
 * ks[0..n_src) is the source sequence, ks[n_src..nk) the target sequence (nk <= 8, at least
 * one kernel each); launches[k] is phase k's launch list (n_launch points, the same parameter
 * n; NULL = sp->launch_src).  Per (launch, seed) each side runs its phases in order on ONE
 * set of global buffers matched by name (pair-level id, X8): a buffer starts from the PRF
 * contents, its size is the largest any phase of the side declares, each phase checks bounds
 * against its own declaration, and a kernel boundary is a grid-wide barrier.  Races / OOB /
 * LIMIT / BARRIER_DIV per phase (record kernel = phase index).  The comparative assertion
 * compares the two sides' final buffers on every id both use and some phase declares out /
 * inout: MISMATCH in kernel 0's slot, tid fields = the last writer in the last phase of the
 * side that declares the buffer out / inout.  Every instance runs in the exact sequential
 * pass (blocks in bid order).  BANK / COALESCE / LOCKSTEP / DATAFLOW are PG_E_ARG. */
int pg_check_equiv_seq(const pg_ir *const *ks, uint32_t nk, uint32_t n_src, const pg_launch *const *launches,
                       const pg_space *sp, pg_run **out);

/* Race premise of the key observation (L516-L520, L660-L662) for one kernel:
 * WW / RW / XB / OOB (and LIMIT) over the space; checks = RACE|OOB regardless
 * of sp->checks. */
int pg_check_races(const pg_ir *k, const pg_space *sp, pg_run **out);

/* Bank-conflict and coalescing conditions (L21-L24, L146-L150; X9) for one
 * kernel; BANK / UNCOALESCED records are failing in this mode.  Per-site
 * statistics are retrievable with pg_collect_site_stats. */
int pg_check_banks(const pg_ir *k, const pg_space *sp, pg_run **out);

/* Property mode: check k
 * against a post-condition given as an IR kernel `post` that computes the expected
 * outputs from the same inputs (the assertion's quantified equalities become its
 * loops; subjects/post_*.pgk).  For launch i, k runs with sp->launch_src[i] and post
 * as one block of one thread whose scalars are the first m (m = post's scalar
 * count) of (gdim.x, gdim.y, bdim.x, bdim.y, launch_src[i].scalar[0..]).  Then the
 * comparative assertion of pg_check_equiv (every out/inout array, matched by name)
 * plus sp->checks on both kernels.  sp->launch_tgt must be NULL (PG_E_ARG); m larger
 * than the available values is PG_E_ARG. */
int pg_check_property(const pg_ir *k, const pg_ir *post, const pg_space *sp, pg_run **out);

/* Synchronise the run's stream, copy the first min(*n_written, cap, max_cex) of the
 * run's OWN records (canonical key order; the run keeps at most pg_space.max_cex,
 * 0 = 2^20) into buf, report how many this run produced in *n_written (may exceed both
 * caps; never the cross-rank total), and fill *sum (may be NULL) from d_first_key /
 * d_counts as they are now - after an all_reduce these are the global summary, so
 * sum->n_records may exceed *n_written. */
int pg_collect_cex(pg_run *r, pg_cex *buf, size_t cap, size_t *n_written, pg_summary *sum);

/* Per-site bank/coalescing statistics of a run: uint64
 * [n_launch][2 kernels][max_sites][8] = [space (1 shared, 2 global), warp
 * accesses, conflicted|uncoalesced, max degree|sectors, sum degree|sectors,
 * sum ideal, sum active lanes, 0]; sites >= max_sites are dropped. */
int pg_collect_site_stats(pg_run *r, uint64_t *buf, uint32_t max_sites);

/* Data-flow relation of a run checked with PG_CHK_DATAFLOW (H5; the bounded form
 * of the fresh-writer instantiation of Fig. 2): one row per in-bounds
 * shared/global read, 12 x uint32 = [launch, seed_idx, block, round, gtid, site,
 * array, addr, src (0 initial, 1 committed write, 2 own write this round),
 * w_block, w_round, w_gtid] (0xFFFFFFFF for initial), in no particular order.
 * *n_rows receives the number of reads (rows beyond the capacity are dropped). */
int pg_collect_dataflow(pg_run *r, uint32_t *rows, size_t cap_rows, size_t *n_rows);

/* Lock-step comparison (X25) of a run checked by
 * pg_check_equiv with PG_CHK_LOCKSTEP: for the shared arrays both kernels declare
 * with the same name and size (and launches with the same number of blocks), the
 * contents after every round < PG_LOCK_ROUNDS of every block are compared.  One row
 * per instance whose shared states diverge, at the first (block, round, array, addr)
 * (array in the source kernel's declaration order): 10 x uint32 = [launch, seed_idx,
 * block, round, array (0x100 + source shared index), addr, val_src, val_tgt,
 * written_src, written_tgt], in (launch, seed) order; *n_rows = their number.
 * Blocks of more than 1024 threads are PG_E_LIMIT in this mode; PG_E_STATE if the run
 * was not checked with PG_CHK_LOCKSTEP. */
int pg_collect_lockstep(pg_run *r, uint32_t *rows, size_t cap_rows, size_t *n_rows);

/* VC-literal cross-check of a run checked with PG_CHK_VCLITERAL:
 * out[0] = reads whose writer was found literally, out[1] = those whose literal writer differs
 * from the data-flow row's owner-stamp writer (0 when the ownership table is right), out[2] =
 * literal scans that met a round beyond the 64 the history keeps.  PG_E_STATE otherwise. */
int pg_collect_vcliteral(pg_run *r, uint64_t out[3]);

/* Introspection of a loaded kernel. */
int pg_ir_info(const pg_ir *k, uint32_t *n_sites, uint32_t *n_globals, uint32_t *n_scalars);
/* *oblivious = 1 when no address, access guard, branch or loop condition of the kernel
 * depends on array contents (no private arrays either): every seed of a launch then takes
 * the same accesses in the same rounds, and the optimistic and exact passes run several
 * seeds per lane (multi-seed lanes); 0 otherwise (e.g. the bitonic
 * compare-exchange, whose store guard depends on the data).  *n_tainted = the variables
 * that may hold an input-dependent value.  PG_E_ARG on a null kernel. */
int pg_ir_seed_oblivious(const pg_ir *k, uint32_t *oblivious, uint32_t *n_tainted);
/* *block_private = 1 when every global array the kernel writes is never loaded and every
 * store to it has the flat index bid.x: distinct blocks of a one-dimensional grid then
 * write distinct cells and read none another block writes, so the cross-block race X4 (XB)
 * cannot occur and checks of such launches skip the XB stamps, K2b and the sequential pass
 * (the SDK reductions' g_odata[bid.x]).  PG_E_ARG on a null kernel. */
int pg_ir_block_private(const pg_ir *k, uint32_t *block_private);
/* *mask bit a (arrays in declaration order) = 1 when array a is a one-dimensional shared
 * array every store of which has the flat index tid.x (or a variable only ever assigned
 * tid.x): in a one-dimensional block no two threads store to one cell, so no WW race on it
 * is possible and its stores take a plain owner stamp instead of a claim (
 * the SDK reductions' sdata[tid]).  PG_E_ARG on a null kernel. */
int pg_ir_thread_private(const pg_ir *k, uint64_t *mask);
/* Generated CUDA source of the evaluation kernel for (bits, checks, bank_model). */
int pg_ir_source(const pg_ir *k, uint32_t bits, uint32_t checks, uint32_t bank_model, char *buf, size_t cap,
                 size_t *len);
/* Compile the evaluation kernel variant now (NVRTC -> sm_100a cubin); no GPU needed. */
int pg_ir_compile(const pg_ir *k, uint32_t bits, uint32_t checks, uint32_t bank_model);

/* Device time of the run's evaluation kernels and of the whole check (CUDA
 * events on the run's stream, ms), the number of CUDA kernels it launched and
 * the host->device bytes it copied (launch tables).  A check whose plan was seen before
 * replays a captured CUDA graph of its body (PGVC_GRAPH=0 disables), so repeated checks
 * enqueue a handful of operations and allocate only their record list. */
int pg_run_timing(pg_run *r, float *ms_eval, float *ms_total, uint32_t *n_launches, uint64_t *h2d_bytes);

/* Start and end (ms) of each of the run's evaluation-kernel launches, as pairs in buf[2i],
 * buf[2i+1], relative to ref_event (a cudaEvent_t recorded before the check, e.g. the
 * caller's step-start event; NULL = the run's first enqueued operation).  The union of
 * these intervals is the evaluation kernel's busy time when launches overlap (the two
 * kernels of a pair run on parallel branches).  *n = number of launches; at most cap pairs
 * are written.  Synchronises the run's stream. */
int pg_run_intervals(pg_run *r, void *ref_event, float *buf, size_t cap, size_t *n);

/* Merge the counters of n_rows checks enqueued on the same device (e.g. the pairs of one
 * step, each with its own rows): d_out_first_key[i] = MIN over rows of d_first_keys[r*11+i],
 * d_out_counts[i] = SUM over rows of d_counts[r*16+i] - the reduction H9 then applies across
 * ranks.  All pointers are device int64 buffers (borrowed); enqueued on `stream`. */
int pg_merge_counters(const int64_t *d_first_keys, const int64_t *d_counts, uint32_t n_rows,
                      int64_t *d_out_first_key, int64_t *d_out_counts, void *stream);

/* Measurement utility (not part of the method; the K2 roofline denominator, SURVEY.md
 * §8(d)): integer ops/s the current device sustains on `stream` for [0] LOP3 chains (alu
 * pipe), [1] IMAD chains (fma pipe), [2] both alternating (the two pipes together).
 * ~50 ms of GPU time; PG_E_CUDA without a device. */
int pg_measure_int32_peak(void *stream, double ops_per_s[3]);

const char *pg_last_error(void);
void pg_ir_free(pg_ir *k);
void pg_run_free(pg_run *r);
const char *pg_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PGVC_H */
