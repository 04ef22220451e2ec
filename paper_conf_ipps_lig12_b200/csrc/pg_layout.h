// pg_layout.h — data layout shared by the host planner (api.cpp) and the
// device runtime (device_rt.cuh, compiled by NVRTC).  Plain C structs only.
#pragma once
#ifndef __CUDACC_RTC__
#include <stdint.h>
#endif

typedef unsigned int u32;
typedef unsigned long long u64;
typedef int i32;
typedef unsigned short u16;

#define PG_FULL 0xffffffffu
#define PG_END 0xFFFFu
#define PG_NEVER 0xFFFFFFFFu
#define PG_NK 10
#define PG_MAXARR 16
#define PG_MAXK 8          // kernels of one check (pg_check_equiv_n)
#define PG_R_INPUT PG_MAXK  // region index of the input region (arenas are regions 0..PG_MAXK-1)

// base pointers of the regions a K1 / K3 job addresses: arena of kernel k, then the input region
struct PgRegions {
    u32* r[PG_MAXK + 1];
};

enum { PGK_BARRIER_DIV = 0, PGK_OOB = 1, PGK_WW = 2, PGK_RW = 3, PGK_XB = 4, PGK_MISMATCH = 5, PGK_BANK = 6,
       PGK_UNCOAL = 7, PGK_UNINIT = 8, PGK_LIMIT = 9 };
enum { PGA_GT = 0, PGA_GI = 1, PGA_SH = 2, PGA_PR = 3 };

// ------------------------------------------------------------------ shared host/device layout
struct PgArr {
    u32 size;       // flat words
    u32 d1, d2;     // trailing dims for the row-major flat index
    u32 kind;       // PGA_*
    u32 rec_id;     // array id in records: gid | 0x100 + slot | 0x200 + slot
    u32 gid;        // pair-level global id (PRF tag, X8)
    u32 flags;      // bit0: reader stamps present (array read and written, race checks on);
                    // bit1: a global array whose stamps live in shared memory (single-block launch)
    // shared arrays (and the stamps of flags-bit-1 global arrays): byte offsets in the group's
    // shared region
    u32 s_val, s_own, s_wmax, s_rmin, s_rmax;
    u32 s_clm;      // claims of the round (exact protocol with claims at store time; s_own then
                    // holds the committed owner only, which loads of the same round consult)
    u32 rsets;      // reader-stamp sets (rmin/rmax hold rsets x size words): 2 when the optimistic
                    // pass checks a round's readers after the next barrier (set = step & 1)
    // global arrays written by the kernel: u32-word offsets in the instance arena
    u64 off_val;    // values
    u64 off_own;    // owner stamp of the last commit: ((2^20-1 - step) << 12) | tid
    u64 off_lw;     // last committing writer (gtid + 1; 0 = initial)
    u64 off_wmax, off_rmin, off_rmax;   // race stamps (~0: absent)
    u64 off_xf, off_xl;                 // first / last accessing block + 1 (~0: absent)
    u64 off_in;     // global arrays the kernel only reads: u32-word offset in the input region
    u64 off_snap;   // lock-step mode, shared arrays matched in the pair: [block][round < R][cell] x
                    // (value, written) word pairs in the instance arena (~0: absent)
};

struct PgLaunchK {
    u32 gdim[3], bdim[3];
    i32 scal[8];
    u32 T, nblocks;
    u32 lpg, gpw, wpg, V, P, cta_threads;
    // per-group shared region: [values | stamps starting at 0 | stamps starting at ~0]
    u32 smem_group_bytes, smem_zero_off, smem_never_off, n_arrays;
    u64 arena_stride, input_stride;          // u32 words per instance
    u64 off_step0;                           // data-flow mode: per-block first round step (arena words), ~0 absent
    u64 off_hist, off_hround;                // VC-literal mode: [block][round < 64][thread][1 + W_max] logged
                                             // writes, [block] rounds (arena words), ~0 absent
    u64 gmag0, gmag01;                       // ceil(2^40 / d) for d = gdim.x and gdim.x * gdim.y: block index ->
                                             // bid by multiply and shift (exact for block indices < 2^20)
    PgArr arr[PG_MAXARR];
};

struct PgWork {
    u32 launch;      // index into the launch table (and the record key)
    u32 ngroups;     // groups in this CTA = seeds x gb
    u32 seed_j0;     // seed index of the item's seed 0
    u32 seed_jstep;  // seed index stride between seeds (= world)
    u32 blk0, blk1;  // emulated blocks [blk0, blk1) of every seed are processed by this CTA
    u32 gb;          // block slots per seed: group g = seed (g / gb), block blk0 + i*gb + (g % gb)
    u32 inst0;       // batch-local instance index of seed 0 (sequential-fallback flags)
    u64 arena_off;   // u32-word offset of seed 0's kernel arena
    u64 input_off;   // u32-word offset of seed 0's input region
    u64 slot0;       // slot index (seed 0, this kernel, kind 0)
    u64 slot_step;   // slot stride between seeds
    u32 nseeds;      // seeds in this item
    u32 item;        // item index (per-item site statistics)
};

struct PgSlot {
    u64 count;
    u32 lock, has;
    u32 f[8];  // round, array, addr, tid_a, tid_b, site, val_a, val_b
    u64 pkey;  // ~(packed prefix of f) of the minimum event, maximised atomically (0: none):
               // a candidate whose packed prefix is larger skips the lock (pg_pack)
};

struct PgParams {
    const PgLaunchK* launches;
    const PgWork* work;
    u32* arena;
    const u32* input;
    PgSlot* slots;
    u64* counts;       // d_counts (int64[16] viewed as u64)
    u64* site_stats;   // parallel pass: [item][max_sites][8]; sequential pass: [n_launch][max_sites][8]
    u32* xb_flag;      // per batch-local instance: some global cell was shared between blocks
    u64 seed_base;
    u32 max_sites;
    u32 kernel_idx;
    u32 fuel;
    u32 seq;           // 0: block-parallel pass; 1: sequential re-run of flagged seed groups;
                       // 2: block-parallel exact re-run of the instances the optimistic pass flagged
    u32 input_mode, input_range, mask;
    u32 count_inst;    // this pass counts instances (X19) into inst_cnt
    u64* inst_cnt;     // per batch-local instance: instances counted (X19), summed by pg_count_reduce
    u32* df_rows;      // data-flow rows (12 words each), PG_CHK_DATAFLOW only
    u32* df_count;
    u32 df_cap;
    u32 pad2;
    const u32* work_list;   // sequential pass: indices (into work) of the items to run
    const u32* work_count;  // their number (device); nullptr: one item per CTA, or
    u32 n_work;             // (non-zero) a grid-stride loop over this many items (exact re-run)
    u32 pad3;
    u32* flag_any;          // set when any instance of the batch is flagged; re-run passes with
                            // nothing flagged exit at once (nullptr: absent)
    u64* op_cnt;            // PG_CHK_OPCOUNT: per batch-local instance, IR integer operations executed
    u32 keep_vals;          // sequential pass of a later phase of a kernel sequence: the global values
                            // are the previous phase's results (only stamps are reset)
    u32 pad4;
    const u32* seq_pref;    // per launch: its instances go straight to the sequential pass (the last
                            // check's sequential pass found an XB race in at least half of them): the
                            // block-parallel passes skip their items, K2b flags them (nullptr: off)
};

// K1 (pg_gen_inputs) job: one buffer of one array for n_inst consecutive
// instances of one launch (instance i at dst + i * stride, seed index j0 + i * jstep).
enum { PGF_CONST = 0, PGF_CELLS = 1, PGF_INPUT = 2 };
struct PgFill {
    u64 dst;      // u32-word offset of instance 0 in the target region
    u64 stride;   // u32 words between instances
    u32 n;        // elements (u32 for CONST/INPUT, u64 cells for CELLS)
    u32 n_inst;
    u32 j0, jstep;
    u32 op;       // PGF_*
    u32 gid;      // PRF tag (X8)
    u32 value;    // PGF_CONST fill value
    u32 target;   // region: arena of kernel k (0..PG_MAXK-1) or PG_R_INPUT
    u32 inst0;    // batch-local index of instance 0 (re-initialisation of flagged instances)
    u32 task0;    // first CTA task of this job in the batch's fill list (pg_fill_tasks)
    u32 istep;    // instances 0, istep, 2 istep, ... (n_inst of them): stamps that only the first
                  // instance of a multi-seed group keeps
    u32 pad;
};
// CTA tasks of a K1 job: a chunk of PG_FILL_CHUNK words of one instance (arrays of more than
// PG_FILL_SMALL words), else 8 instances (a warp each)
#define PG_FILL_CHUNK 16384u
#define PG_FILL_SMALL 512u
#ifndef __CUDACC_RTC__
static inline u32 pg_fill_tasks(u32 n, u32 n_inst) {
    return n > PG_FILL_SMALL ? n_inst * ((n + PG_FILL_CHUNK - 1u) / PG_FILL_CHUNK) : (n_inst + 7u) / 8u;
}
#endif

// K2b (pg_xb_detect) job: one global array written by a kernel, for n_inst
// consecutive instances of one launch: flags instances whose cells were
// accessed by two blocks with a committed write (X4 XB).
struct PgXb {
    u64 xf, xl, lw;   // u32-word offsets of instance 0 in the kernel arena
    u64 stride;
    u32 n, n_inst, inst0;
    u32 istep;        // multi-seed launches: the marks live in the first instance of each group of
                      // istep seeds, whose verdict holds for the whole group
    u32 task0;        // first CTA task (pg_fill_tasks over the instances holding marks)
    u32 launch;       // the launch (index into the launch table) of the job's instances
};

// K3b (pg_lockstep) job: one shared array both kernels of a pair declare (same name
// and size), snapshotted after rounds < R of every block, for n_inst instances.
struct PgLock {
    u64 src_off, tgt_off;        // u32-word offsets of instance 0's snapshots in the two arenas
    u64 src_stride, tgt_stride;  // arena strides
    u64 key0;                    // index of instance 0 in the run's per-instance tables
    u32 n_inst, nblocks, size, rounds, arr_slot, pad;
};

// K3 (pg_compare) job: one global array (pair-level id) of one launch segment, compared
// between every pair of the kernels that have it (H7): member m is kernel kid[m]'s copy.  A
// pair (a, b), a < b, is compared when pair_mask has bit a * PG_MAXK + b (one of the two
// declares it out / inout), on the cells below both declared sizes; its mismatches are
// events of kernel kid[a]'s MISMATCH slot.  Each cell is read once per member, not once per
// pair.
struct PgCmp {
    u64 off[PG_MAXK];            // value words of instance 0 in the member's region
    u64 stride[PG_MAXK];         // per-instance stride of that region
    u64 lw[PG_MAXK];             // last-writer words of instance 0 (members with bit m of lw_flags)
    u32 region[PG_MAXK];         // arena of kernel k, or PG_R_INPUT (array only read)
    u32 size[PG_MAXK];           // the member's declared size
    u32 kid[PG_MAXK];            // the member's kernel index (record slot)
    u32 lwg[PG_MAXK];            // multi-seed group of the member's launch: its last-writer words live
                                 // in the group's first instance (the same cells in every seed)
    u64 pair_mask;
    u64 slot0, slot_step;        // MISMATCH slot of (instance 0, kernel 0) and the instance stride
    u64 mm0, mm_step;            // min-cell words of (instance 0, kernel 0) and the instance stride
    u32 inst0, n_inst, gid, n;   // n: cells scanned (the largest member size)
    u32 nm;                      // members
    u32 lw_flags;
    u32 nmode;                   // N-kernel check: record site = the other kernel; else PG_NEVER
    u32 task0;                   // first CTA task (pg_fill_tasks(n, n_inst))
    u32 pad_writes_;             // (planner scratch: members that declare the array out / inout)
    u32 pad_;
};
