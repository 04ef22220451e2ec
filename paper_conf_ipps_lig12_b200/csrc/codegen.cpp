// codegen.cpp — IR -> CUDA C++ of the evaluation kernel (K2).
//
// The kernel body becomes a re-entrant "segment" function: each call runs one
// emulated thread from its resume point to the next barrier (`return k`) or to
// the end (`return PG_END`); the runtime (device_rt.cuh) performs the round
// protocol between calls.  Control flow follows the uniformity analysis:
//   * block-uniform if / loop  -> real branches (gotos at function top level,
//     so a barrier inside a uniform loop is simply a resume label);
//   * thread-dependent if / loop -> if-converted with per-lane predicates
//     and warp-uniform `__any_sync` skips, so every lane of a warp executes
//     every access site together (the lock-step warp access of X9) and the
//     warp-level bank / coalescing intrinsics see the whole warp.
// Loads are predicated (short-circuit && || ?: keep their guards, X2/X21).
#include <cstdio>
#include <map>
#include <set>
#include <sstream>

#include "front.hpp"

namespace pgf {

namespace {

std::string hex(uint32_t v) {
    char b[16];
    std::snprintf(b, sizeof b, "0x%08xu", v);
    return b;
}

// ---------------------------------------------------------------- seed-oblivious analysis
// Input dependence ("taint"): a load's value depends on the seed; so does every expression
// over it and every variable assigned one (fixed point).  The kernel is seed-oblivious when
// no address, store guard, branch or loop condition is tainted: then all seeds of a launch
// take the same accesses in the same rounds (the stamps, races and instance counts agree)
// and one lane can carry several seeds' values (multi-seed lanes).
struct Taint {
    std::vector<bool> tv;
    bool ok = true;
    bool tainted(const Node* n) const {
        if (!n) return false;
        if (n->kind == NK::Elem) return true;
        if (n->kind == NK::Var) return tv[(size_t)n->ref];
        for (const Node* k : n->kids)
            if (tainted(k)) return true;
        return false;
    }
    static bool has_load(const Node* n) {
        if (!n) return false;
        if (n->kind == NK::Elem) return true;
        for (const Node* k : n->kids)
            if (has_load(k)) return true;
        return false;
    }
    bool prop(const Stmt* s) {
        if (!s) return false;
        bool ch = false;
        switch (s->kind) {
        case SK::Seq:
            for (const Stmt* c : s->seq) ch |= prop(c);
            break;
        case SK::Assign:
            if (!tv[(size_t)s->var] && tainted(s->value)) tv[(size_t)s->var] = ch = true;
            break;
        case SK::If: ch |= prop(s->body); ch |= prop(s->other); break;
        case SK::Loop: ch |= prop(s->init); ch |= prop(s->body); ch |= prop(s->step); break;
        default: break;
        }
        return ch;
    }
    void check_expr(const Node* n) {
        if (!n) return;
        if (n->kind == NK::Elem)
            for (const Node* i : n->kids)
                if (tainted(i)) ok = false;   // input-dependent address
        if ((n->kind == NK::LAnd || n->kind == NK::LOr || n->kind == NK::Select) && tainted(n->kids[0]))
            for (size_t i = 1; i < n->kids.size(); i++)
                if (has_load(n->kids[i])) ok = false;   // input-dependent load guard
        for (const Node* k : n->kids) check_expr(k);
    }
    void check(const Stmt* s) {
        if (!s) return;
        switch (s->kind) {
        case SK::Seq:
            for (const Stmt* c : s->seq) check(c);
            break;
        case SK::Assign: check_expr(s->value); break;
        case SK::Store:
            for (const Node* i : s->index) {
                if (tainted(i)) ok = false;
                check_expr(i);
            }
            check_expr(s->value);
            break;
        case SK::PrivDecl: ok = false; break;
        case SK::If:
            if (tainted(s->cond)) ok = false;   // input-dependent guard of the branches' accesses
            check_expr(s->cond);
            check(s->body);
            check(s->other);
            break;
        case SK::Loop:
            check(s->init);
            if (tainted(s->cond)) ok = false;
            check_expr(s->cond);
            check(s->body);
            check(s->step);
            break;
        default: break;
        }
    }
};

struct Gen {
    const Kernel& K;
    const CodegenOptions& O;
    uint32_t mask;
    std::ostringstream body;
    int ntmp = 0, nlabel = 0, nsync = 0;
    std::vector<uint32_t> sync_sites_;   // site of each seg() resume point, in order

    struct Loop {
        int id;
        bool uniform;
        std::string act;      // non-uniform: active-lane predicate
        size_t body_depth;    // non-uniform: predicate-stack index of the body predicate
        int cont_label = -1, exit_label = -1;
    };
    std::vector<std::string> preds;  // thread-dependent predicate variables, innermost last
    std::vector<Loop> loops;
    std::vector<bool> log_;          // per array: a load may follow the thread's own store in one round
    bool inline_ = false;            // emitting `run` (rounds inline) rather than the re-entrant `seg`

    // ---------------------------------------------------------------- own-write analysis
    // Conservative flow walk: which arrays may have been stored by this thread since
    // the last barrier?  A load of such an array must consult the write log (X3);
    // others read memory directly.
    void lw_expr(const Node* n, const std::vector<bool>& stored) {
        if (!n) return;
        for (const Node* k : n->kids) lw_expr(k, stored);
        if (n->kind == NK::Elem && stored[(size_t)n->ref]) log_[(size_t)n->ref] = true;
    }
    void lw_stmt(const Stmt* s, std::vector<bool>& st) {
        if (!s) return;
        switch (s->kind) {
        case SK::Seq:
            for (const Stmt* c : s->seq) lw_stmt(c, st);
            break;
        case SK::Assign: lw_expr(s->value, st); break;
        case SK::Store:
            for (const Node* i : s->index) lw_expr(i, st);
            lw_expr(s->value, st);
            st[(size_t)s->arr] = true;
            break;
        case SK::Sync: std::fill(st.begin(), st.end(), false); break;
        case SK::If: {
            lw_expr(s->cond, st);
            std::vector<bool> a = st, b = st;
            lw_stmt(s->body, a);
            lw_stmt(s->other, b);
            for (size_t i = 0; i < st.size(); i++) st[i] = a[i] || b[i];
            break;
        }
        case SK::Loop: {
            lw_stmt(s->init, st);
            for (int pass = 0; pass < 3; pass++) {  // a store can reach a load of the next iteration
                std::vector<bool> in = st;
                lw_expr(s->cond, in);
                lw_stmt(s->body, in);
                lw_stmt(s->step, in);
                for (size_t i = 0; i < st.size(); i++) st[i] = st[i] || in[i];
            }
            lw_expr(s->cond, st);
            break;
        }
        default: break;
        }
    }

    // ---------------------------------------------------------------- round-segment analysis
    // Barriers are block-uniform (X18), so in one round every thread of a block runs code
    // entered from the same barrier.  For each program point: the set of barriers (nullptr =
    // kernel entry) from which it is reachable without crossing another barrier.  A load of
    // an array needs reader stamps only if some store to that array shares a barrier with
    // it: otherwise no write of the array can fall in the load's round (no RW race, X4).
    using SegSet = std::set<const Stmt*>;
    std::map<const Node*, SegSet> seg_ld_;
    std::vector<SegSet> seg_st_;
    bool seg_changed_ = false;
    static bool merge_into(SegSet& dst, const SegSet& src) {
        size_t n = dst.size();
        dst.insert(src.begin(), src.end());
        return dst.size() != n;
    }
    void seg_expr(const Node* n, const SegSet& st) {
        if (!n) return;
        for (const Node* k : n->kids) seg_expr(k, st);
        if (n->kind == NK::Elem) seg_changed_ |= merge_into(seg_ld_[n], st);
    }
    void seg_stmt(const Stmt* s, SegSet& st) {
        if (!s) return;
        switch (s->kind) {
        case SK::Seq:
            for (const Stmt* c : s->seq) seg_stmt(c, st);
            break;
        case SK::Assign: seg_expr(s->value, st); break;
        case SK::Store:
            for (const Node* i : s->index) seg_expr(i, st);
            seg_expr(s->value, st);
            seg_changed_ |= merge_into(seg_st_[(size_t)s->arr], st);
            break;
        case SK::PrivDecl:
            for (const Node* i : s->index) seg_expr(i, st);
            seg_expr(s->value, st);
            break;
        case SK::Sync: st = SegSet{s}; break;
        case SK::If: {
            seg_expr(s->cond, st);
            SegSet a = st, b = st;
            seg_stmt(s->body, a);
            seg_stmt(s->other, b);
            st = a;
            merge_into(st, b);
            break;
        }
        case SK::Loop: {
            // conservative: the head sees its entry and every state inside the loop (covers
            // back edges, continue and break); iterate to a fixed point
            seg_stmt(s->init, st);
            SegSet head = st;
            for (;;) {
                SegSet in = head, all = head;
                seg_expr(s->cond, in);
                seg_stmt(s->body, in);
                merge_into(all, in);
                seg_stmt(s->step, in);
                merge_into(all, in);
                if (!merge_into(head, all)) break;
            }
            seg_expr(s->cond, head);
            st = head;
            break;
        }
        default: break;
        }
    }
    void seg_run() {
        seg_st_.assign(K.arrays.size(), SegSet());
        do {
            seg_changed_ = false;
            SegSet st{nullptr};
            seg_stmt(K.body, st);
        } while (seg_changed_);
    }
    // reader stamps for this load site
    bool stamps_needed(const Node* n) const {
        if (!reader_tracked(n->ref)) return false;
        if (K.div_barrier) return true;   // (threads of one round may have entered from different barriers)
        auto it = seg_ld_.find(n);
        if (it == seg_ld_.end()) return true;
        for (const Stmt* b : it->second)
            if (seg_st_[(size_t)n->ref].count(b)) return true;
        return false;
    }

    Gen(const Kernel& k, const CodegenOptions& o) : K(k), O(o) {
        mask = o.bits >= 32 ? 0xFFFFFFFFu : ((1u << o.bits) - 1u);
        tidv_ = tid_alias_vars(k);
        tpa_ = thread_private_stores(k);
    }
    // optimistic pass: a load of a thread-private array at index tid.x reads the cell only its
    // own thread writes - it cannot be half of a RW race, so (when the launch's block is 1-D,
    // PgSA::tp) it takes no reader stamp.  The exact protocol keeps every reader stamp: X16's
    // RW record takes the minimum / maximum reader over all of them.
    std::vector<bool> tidv_, tpa_;
    bool self_load(const Node* n) const {
        if (!O.fast || n->kids.size() != 1 || !tpa_[(size_t)n->ref]) return false;
        const Node* ix = n->kids[0];
        while (ix && ix->kind == NK::Cast && ix->kids.size() == 1) ix = ix->kids[0];
        return ix && ((ix->kind == NK::Builtin && ix->ref == 0) ||
                      (ix->kind == NK::Var && ix->ref >= 0 && tidv_[(size_t)ix->ref]));
    }

    std::string tmp(const char* p = "t") { return std::string("_") + p + std::to_string(ntmp++); }

    // ---------------------------------------------------------------- multi-seed lanes
    // (O.ms > 1) tainted values are arrays of PG_MS words, one per seed; untainted ones
    // (addresses, guards, loop counters) stay scalar and are computed once for all seeds
    std::vector<bool> tvar_;
    std::set<std::string> tnames_;   // temporaries / frame slots holding PG_MS copies
    bool ms() const { return O.ms > 1; }
    bool tn(const std::string& x) const { return ms() && tnames_.count(x) != 0; }
    std::string at(const std::string& x) const { return tn(x) ? x + "[_s]" : x; }
    std::string defv(const std::string& e) {   // e refers to its operands through at()
        std::string r = tmp();
        line("u32 " + r + "[PG_MS]; PG_S_LOOP " + r + "[_s] = " + e + ";");
        tnames_.insert(r);
        return r;
    }
    std::string def2(bool t, const std::string& e) { return t ? defv(e) : def(e); }
    std::string vec(const std::string& x) {   // a PG_MS-word copy of x (store operands)
        if (tn(x)) return x;
        return defv(x);
    }
    int label() { return nlabel++; }
    void line(const std::string& s) { body << "  " << s << "\n"; }
    bool uniform_ctx() const { return preds.empty(); }
    std::string cur() const { return preds.empty() ? std::string("1u") : preds.back(); }
    std::string eff() const { return preds.empty() ? std::string("t.live") : "(" + preds.back() + " & t.live)"; }

    // reader stamps: race checks on, or the optimistic pass (which must detect every race)
    bool reader_tracked(int arr) const {
        const ArrayDecl& a = K.arrays[(size_t)arr];
        return ((O.checks & PG_RACE_BIT) || O.fast) && a.written && a.read && a.space != PRIVATE;
    }
    // optimistic pass: a store of the array must look for readers of its round
    std::vector<bool> rda_;
    std::string rda(int arr) const { return O.fast && rda_[(size_t)arr] ? "true" : "false"; }
    static constexpr uint32_t PG_RACE_BIT = 2;

    uint32_t priv_size(const ArrayDecl& a) const {
        uint64_t s = 1;
        for (const Node* d : a.dims) s *= d->lit;
        return (uint32_t)s;
    }

    // ---------------------------------------------------------------- expressions
    // PG_CHK_OPCOUNT: count one IR integer operation executed under predicate pr
    void opc(const std::string& pr, int n = 1) {
        if (O.checks & 128) line("t.ops += " + std::to_string(n) + "u * (u32)(" + pr + ");");
    }
    std::string flat_index(const Node* n, int arr, const std::string& pr) {
        std::vector<std::string> iv;
        for (const Node* k : n->kids) iv.push_back(ex(k, pr));
        const ArrayDecl& a = K.arrays[(size_t)arr];
        std::string f = tmp("f");
        line("u32 " + f + " = " + iv[0] + ";");
        for (size_t k = 1; k < iv.size(); k++) {
            std::string dim;
            if (a.space == PRIVATE) dim = hex(a.dims[k]->lit);
            else if (a.space == SHARED) dim = "PG_SH(" + std::to_string(arr) + ", d" + std::to_string(k) + ")";
            else dim = "pg_sL.arr[" + std::to_string(arr) + "].d" + std::to_string(k);
            line(f + " = " + f + " * " + dim + " + " + iv[k] + ";");
            opc(pr, 2);   // (row-major flattening: a multiply and an add per extra dimension)
        }
        return f;
    }
    std::string ex(const Node* n, const std::string& pr) {
        switch (n->kind) {
        case NK::Neg: case NK::BitNot: case NK::LogNot: case NK::Bin: case NK::LAnd: case NK::LOr:
        case NK::Select: case NK::Min: case NK::Max:
            opc(pr);
            break;
        default:
            break;
        }
        switch (n->kind) {
        case NK::Lit: return hex(n->lit & mask);
        case NK::Var: return "F.v" + std::to_string(n->ref);
        case NK::Builtin: {
            int c = n->ref % 3;
            std::string src;
            if (n->ref < 3) src = "t.tid[" + std::to_string(c) + "]";
            else if (n->ref < 6) src = "t.bid[" + std::to_string(c) + "]";
            else if (n->ref < 9) src = "PG_BDIM" + std::to_string(c);
            else src = "pg_sL.gdim[" + std::to_string(c) + "]";
            return "pg_m(" + src + ")";
        }
        case NK::Elem: {
            const ArrayDecl& a = K.arrays[(size_t)n->ref];
            std::string f = flat_index(n, n->ref, pr);
            std::string r = tmp();
            std::string A = std::to_string(n->ref), S = std::to_string(n->site) + "u";
            const std::string st = !stamps_needed(n) ? "false" : self_load(n) ? "!PG_TP_CONST(" + A + ")" : "true";
            const std::string lg = log_[(size_t)n->ref] ? "true" : "false";
            if (ms()) {   // (seed-oblivious: shared or global, never private)
                line("u32 " + r + "[PG_MS];");
                tnames_.insert(r);
                if (a.space == SHARED)
                    line("pg_ld_sh_ms<" + A + ", " + st + ", " + lg + ">(C, t, c, ss, " + pr + ", " + f + ", " + S + ", " + r + ");");
                else if (a.written)
                    line("pg_ld_gt_ms<" + A + ", " + st + ", " + lg + ">(C, t, c, ss, " + pr + ", " + f + ", " + S + ", " + r + ");");
                else
                    line("pg_ld_gi_ms<" + A + ">(C, t, c, ss, " + pr + ", " + f + ", " + S + ", " + r + ");");
                return r;
            }
            if (a.space == SHARED) {
                line("u32 " + r + " = pg_ld_sh<" + A + ", " + st + ", " + lg + ">(C, t, c, ss, " + pr + ", " + f + ", " + S + ");");
            } else if (a.space == GLOBAL) {
                if (a.written)
                    line("u32 " + r + " = pg_ld_gt<" + A + ", " + st + ", " + lg + ">(C, t, c, ss, " + pr + ", " + f + ", " + S + ");");
                else
                    line("u32 " + r + " = pg_ld_gi<" + A + ">(C, t, c, ss, " + pr + ", " + f + ", " + S + ");");
            } else {
                line("u32 " + r + " = pg_priv_ok(C, t, c, " + pr + ", " + f + ", " + hex(priv_size(a)) + ", " +
                     hex(0x200u + (uint32_t)a.slot) + ", " + S + ", 0u, 0u) ? F.p" + std::to_string(a.slot) + "[" +
                     f + "] : 0u;");
            }
            return r;
        }
        case NK::Neg: { std::string a = ex(n->kids[0], pr); return def2(tn(a), "pg_neg(" + at(a) + ")"); }
        case NK::BitNot: { std::string a = ex(n->kids[0], pr); return def2(tn(a), "pg_not(" + at(a) + ")"); }
        case NK::LogNot: { std::string a = ex(n->kids[0], pr); return def2(tn(a), "(u32)(" + at(a) + " == 0u)"); }
        case NK::Cast: return ex(n->kids[0], pr);
        case NK::LAnd:
        case NK::LOr: {
            const bool land = n->kind == NK::LAnd;
            std::string x = ex(n->kids[0], pr);
            std::string a = def2(tn(x), "(u32)(" + at(x) + " != 0u)");
            if (tn(a)) {   // input-dependent condition: the other operand has no loads (seed_oblivious)
                std::string b = ex(n->kids[1], pr);
                return defv(at(a) + (land ? " & " : " | ") + "(u32)(" + at(b) + " != 0u)");
            }
            std::string p = def(land ? "(" + pr + ") & " + a : "(" + pr + ") & (" + a + " ^ 1u)");
            std::string b = ex(n->kids[1], p);
            return def2(tn(b), a + (land ? " & " : " | ") + "(u32)(" + at(b) + " != 0u)");
        }
        case NK::Select: {
            std::string cx = ex(n->kids[0], pr);
            std::string c = def2(tn(cx), "(u32)(" + at(cx) + " != 0u)");
            if (tn(c)) {
                std::string x = ex(n->kids[1], pr), y = ex(n->kids[2], pr);
                return defv(at(c) + " ? " + at(x) + " : " + at(y));
            }
            std::string p1 = def("(" + pr + ") & " + c);
            std::string p0 = def("(" + pr + ") & (" + c + " ^ 1u)");
            std::string x = ex(n->kids[1], p1);
            std::string y = ex(n->kids[2], p0);
            return def2(tn(x) || tn(y), c + " ? " + at(x) + " : " + at(y));
        }
        case NK::Min:
        case NK::Max: {
            std::string a0 = ex(n->kids[0], pr), b0 = ex(n->kids[1], pr);
            const bool T = tn(a0) || tn(b0);
            std::string a = at(a0), b = at(b0);
            std::string lt = n->opty == Ty::U32 ? "(" + a + " < " + b + ")" : "pg_slt(" + a + ", " + b + ")";
            return def2(T, n->kind == NK::Min ? lt + " ? " + a + " : " + b : lt + " ? " + b + " : " + a);
        }
        case NK::Bin: {
            std::string a0 = ex(n->kids[0], pr), b0 = ex(n->kids[1], pr);
            const bool T = tn(a0) || tn(b0);
            std::string a = at(a0), b = at(b0);
            bool u = n->opty == Ty::U32;
            switch (n->op) {
            case Bop::Add: return def2(T, "pg_add(" + a + ", " + b + ")");
            case Bop::Sub: return def2(T, "pg_sub(" + a + ", " + b + ")");
            case Bop::Mul: return def2(T, "pg_mul(" + a + ", " + b + ")");
            case Bop::Div: return def2(T, std::string(u ? "pg_udiv(" : "pg_sdiv(") + a + ", " + b + ")");
            case Bop::Rem: return def2(T, std::string(u ? "pg_urem(" : "pg_srem(") + a + ", " + b + ")");
            case Bop::Shl: return def2(T, "pg_shl(" + a + ", " + b + ")");
            case Bop::Shr: return def2(T, std::string(u ? "pg_lshr(" : "pg_ashr(") + a + ", " + b + ")");
            case Bop::And: return def2(T, "(" + a + " & " + b + ")");
            case Bop::Or: return def2(T, "(" + a + " | " + b + ")");
            case Bop::Xor: return def2(T, "(" + a + " ^ " + b + ")");
            case Bop::Lt: return def2(T, u ? "(u32)(" + a + " < " + b + ")" : "pg_slt(" + a + ", " + b + ")");
            case Bop::Le: return def2(T, u ? "(u32)(" + a + " <= " + b + ")" : "pg_sle(" + a + ", " + b + ")");
            case Bop::Gt: return def2(T, u ? "(u32)(" + a + " > " + b + ")" : "pg_slt(" + b + ", " + a + ")");
            case Bop::Ge: return def2(T, u ? "(u32)(" + a + " >= " + b + ")" : "pg_sle(" + b + ", " + a + ")");
            case Bop::Eq: return def2(T, "(u32)(" + a + " == " + b + ")");
            case Bop::Ne: return def2(T, "(u32)(" + a + " != " + b + ")");
            }
        }
        }
        return "0u";
    }
    std::string def(const std::string& e) {
        std::string r = tmp();
        line("const u32 " + r + " = " + e + ";");
        return r;
    }

    // ---------------------------------------------------------------- statements
    void kill_preds(const std::string& k, size_t down_to) {
        for (size_t i = preds.size(); i-- > down_to;) line(preds[i] + " &= " + k + " ^ 1u;");
    }
    void stmt(const Stmt* s) {
        switch (s->kind) {
        case SK::Seq:
            for (const Stmt* c : s->seq) stmt(c);
            return;
        case SK::Nop: return;
        case SK::Assign: {
            line("{");
            std::string v = ex(s->value, eff());
            std::string dst = "F.v" + std::to_string(s->var);
            if (tn(dst)) {
                if (uniform_ctx()) line("PG_S_LOOP " + dst + "[_s] = " + at(v) + ";");
                else line("PG_S_LOOP " + dst + "[_s] = " + eff() + " ? " + at(v) + " : " + dst + "[_s];");
            } else if (uniform_ctx()) {
                line(dst + " = " + v + ";");
            } else {
                line(dst + " = " + eff() + " ? " + v + " : " + dst + ";");
            }
            line("}");
            return;
        }
        case SK::Store: {
            line("{");
            const ArrayDecl& a = K.arrays[(size_t)s->arr];
            Node tmpn;
            tmpn.kids = s->index;
            std::string pe = eff();
            std::string f = flat_index(&tmpn, s->arr, pe);
            std::string v = ex(s->value, pe);
            std::string A = std::to_string(s->arr), S = std::to_string(s->site) + "u";
            if (ms()) {
                v = vec(v);
                line(std::string(a.space == SHARED ? "pg_st_sh_ms<" : "pg_st_gt_ms<") + A + ", " + rda(s->arr) +
                     ">(C, t, c, ss, " + pe + ", " + f + ", " + v + ", " + S + ");");
                line("}");
                return;
            }
            if (a.space == SHARED)
                line("pg_st_sh<" + A + ", " + rda(s->arr) + ">(C, t, c, ss, " + pe + ", " + f + ", " + v + ", " + S + ");");
            else if (a.space == GLOBAL)
                line("pg_st_gt<" + A + ", " + rda(s->arr) + ">(C, t, c, ss, " + pe + ", " + f + ", " + v + ", " + S + ");");
            else
                line("if (pg_priv_ok(C, t, c, " + pe + ", " + f + ", " + hex(priv_size(a)) + ", " +
                     hex(0x200u + (uint32_t)a.slot) + ", " + S + ", " + v + ", 1u)) F.p" + std::to_string(a.slot) +
                     "[" + f + "] = " + v + ";");
            line("}");
            return;
        }
        case SK::PrivDecl: {
            const ArrayDecl& a = K.arrays[(size_t)s->arr];
            std::string pe = eff();
            line("if (" + pe + ") { for (u32 _i = 0; _i < " + hex(priv_size(a)) + "; _i++) F.p" +
                 std::to_string(a.slot) + "[_i] = 0u; }");
            return;
        }
        // (a kernel with a barrier under thread-dependent control runs every branch as a
        // per-thread branch: each thread stops at its own barrier, X18)
        case SK::If:
            if (s->uniform || K.div_barrier) uniform_if(s);
            else predicated_if(s);
            return;
        case SK::Loop:
            if (s->uniform || K.div_barrier) uniform_loop(s);
            else predicated_loop(s);
            return;
        case SK::Sync: {
            int k = ++nsync;
            if (!inline_) sync_sites_.push_back((uint32_t)s->site);
            if (inline_) {   // end this round in place; stop when every thread has exited
                line("if (!pg_round_end<PgK, false>(C, t, c, ar)) return;");
                return;
            }
            line("return " + std::to_string(k) + "u;");
            body << "R" << k << ":;\n";
            return;
        }
        case SK::Return:
            if (uniform_ctx()) {
                line(inline_ ? "t.live = 0u; goto PG_DONE;" : "t.live = 0u; return PG_END;");
            } else {
                line("{");
                line("const u32 _k = " + eff() + ";");
                line("t.live &= _k ^ 1u;");
                kill_preds("_k", 0);
                line("}");
            }
            return;
        case SK::Break:
        case SK::Continue: {
            const Loop& L = loops.back();
            if (L.uniform) {
                line("goto L" + std::to_string(s->kind == SK::Break ? L.exit_label : L.cont_label) + ";");
                return;
            }
            line("{");
            line("const u32 _k = " + eff() + ";");
            if (s->kind == SK::Break) line(L.act + " &= _k ^ 1u;");
            kill_preds("_k", L.body_depth);
            line("}");
            return;
        }
        }
    }
    void uniform_if(const Stmt* s) {
        int le = label(), lend = label();
        line("{");
        std::string c = ex(s->cond, "t.live");
        line("if (!" + c + ") goto L" + std::to_string(le) + ";");
        line("}");
        stmt(s->body);
        if (s->other) line("goto L" + std::to_string(lend) + ";");
        body << "L" << le << ":;\n";
        if (s->other) {
            stmt(s->other);
            body << "L" << lend << ":;\n";
        }
    }
    void predicated_if(const Stmt* s) {
        line("{");
        std::string c = ex(s->cond, eff());
        std::string pt = tmp("p"), pf = tmp("p");
        line("u32 " + pt + " = " + cur() + " & (u32)(" + c + " != 0u);");
        line("u32 " + pf + " = " + cur() + " & (u32)(" + c + " == 0u);");
        line("if (__any_sync(PG_FULL, " + pt + " & t.live)) {");
        preds.push_back(pt);
        stmt(s->body);
        preds.pop_back();
        line("}");
        if (s->other) {
            line("if (__any_sync(PG_FULL, " + pf + " & t.live)) {");
            preds.push_back(pf);
            stmt(s->other);
            preds.pop_back();
            line("}");
        }
        line("}");
    }
    // ---------------------------------------------------------------- fuel (X19)
    static bool has_kind(const Stmt* s, SK k) {
        if (!s) return false;
        if (s->kind == k) return true;
        for (const Stmt* x : s->seq)
            if (has_kind(x, k)) return true;
        return has_kind(s->body, k) || has_kind(s->other, k) || has_kind(s->init, k) ||
               has_kind(s->step, k);
    }
    // The back-edge of a loop whose body passes its last top-level barrier on every
    // path to the back-edge (no `continue` before that barrier), with no loop after
    // the barrier or in the step, is the first back-edge of its round: the round began
    // at that barrier.  Its fuel count (1) cannot exceed the limit, so only the
    // counters advance (same counts as pg_tick; the check is dropped).
    static bool first_backedge_of_round(const Stmt* s) {
        const Stmt* b = s->body;
        if (!b || has_kind(s->step, SK::Loop)) return false;
        if (b->kind == SK::Sync) return true;
        if (b->kind != SK::Seq) return false;
        int last = -1;
        for (size_t i = 0; i < b->seq.size(); i++)
            if (b->seq[i]->kind == SK::Sync) last = (int)i;
        if (last < 0) return false;
        for (int i = 0; i < last; i++)
            if (has_kind(b->seq[i], SK::Continue)) return false;
        for (size_t i = last + 1; i < b->seq.size(); i++)
            if (has_kind(b->seq[i], SK::Loop)) return false;
        return true;
    }
    void uniform_loop(const Stmt* s) {
        const bool fuel_free = first_backedge_of_round(s);
        if (s->init) stmt(s->init);
        Loop L;
        L.id = s->loop;
        L.uniform = true;
        int head = label();
        L.cont_label = label();
        L.exit_label = label();
        body << "L" << head << ":;\n";
        if (s->cond) {
            line("{");
            std::string c = ex(s->cond, "t.live");
            line("if (!" + c + ") goto L" + std::to_string(L.exit_label) + ";");
            line("}");
        }
        loops.push_back(L);
        stmt(s->body);
        body << "L" << L.cont_label << ":;\n";
        if (s->step) stmt(s->step);
        loops.pop_back();
        if (fuel_free) {
            line("t.fuel += (t.live != 0u); ++C.ufuel;");
        } else {
            line("pg_tick(C, t, c, t.live);");
            line(inline_ ? "if (++C.ufuel > C.fuel) { t.live = 0u; goto PG_DONE; }"
                         : "if (++C.ufuel > C.fuel) { t.live = 0u; return PG_END; }");
        }
        line("goto L" + std::to_string(head) + ";");
        body << "L" << L.exit_label << ":;\n";
    }
    void predicated_loop(const Stmt* s) {
        if (s->init) stmt(s->init);
        line("{");
        Loop L;
        L.id = s->loop;
        L.uniform = false;
        L.act = tmp("a");
        line("u32 " + L.act + " = " + cur() + ";");
        line("for (;;) {");
        if (s->cond) {
            line("{");
            std::string c = ex(s->cond, "(" + L.act + " & t.live)");
            line(L.act + " &= (u32)(" + c + " != 0u);");
            line("}");
        }
        line(L.act + " &= t.live;");
        line("if (!__any_sync(PG_FULL, " + L.act + ")) break;");
        std::string b = tmp("b");
        line("{");
        line("u32 " + b + " = " + L.act + ";");
        preds.push_back(b);
        L.body_depth = preds.size() - 1;
        loops.push_back(L);
        stmt(s->body);
        loops.pop_back();
        preds.pop_back();
        line("}");
        if (s->step) {
            preds.push_back(L.act);
            stmt(s->step);
            preds.pop_back();
        }
        line("pg_tick(C, t, c, " + L.act + " & t.live);");
        line("}");
        line("}");
    }

    std::string run() {
        log_.assign(K.arrays.size(), false);
        {
            std::vector<bool> st(K.arrays.size(), false);
            lw_stmt(K.body, st);
        }
        seg_run();
        tvar_.assign(K.vars.size(), false);
        if (ms()) {
            if (!seed_oblivious(K, &tvar_)) throw FrontError(-7, "multi-seed variant of a kernel that is not seed-oblivious");
            for (size_t i = 0; i < K.vars.size(); i++)
                if (tvar_[i]) tnames_.insert("F.v" + std::to_string(i));
        }
        rda_.assign(K.arrays.size(), false);
        for (const auto& ld : seg_ld_)
            if (stamps_needed(ld.first)) rda_[(size_t)ld.first->ref] = true;
        // the body twice: `seg` (re-entrant at every barrier; virtual-thread variants) and
        // `run` (a whole block, rounds ended in place)
        auto emit = [&](bool inl) {
            ntmp = nlabel = nsync = 0;
            sync_sites_.clear();
            body.str("");
            preds.clear();
            loops.clear();
            inline_ = inl;
            stmt(K.body);
            if (inl) {
                line("t.live = 0u;");
                body << "PG_DONE:;\n";
                line("pg_round_end<PgK, true>(C, t, c, ar);");
            } else {
                line("t.live = 0u; return PG_END;");
            }
            return body.str();
        };
        const std::string seg_body = emit(false);
        const int seg_nsync = nsync;
        const std::vector<uint32_t> seg_sites = sync_sites_;
        const std::string run_body = emit(true);
        std::ostringstream o;
        o << "#define PG_BITS " << O.bits << "\n";
        o << "#define PG_RACECHK " << ((O.checks & 2) ? 1 : 0) << "\n";
        o << "#define PG_OOBCHK " << ((O.checks & 4) ? 1 : 0) << "\n";
        o << "#define PG_BANKCHK " << ((O.checks & 8) ? 1 : 0) << "\n";
        o << "#define PG_COALCHK " << ((O.checks & 16) ? 1 : 0) << "\n";
        o << "#define PG_BANK16 " << (O.bank_model == 1 ? 1 : 0) << "\n";
        o << "#define PG_DATAFLOW " << ((O.checks & 32) ? 1 : 0) << "\n";
        o << "#define PG_LOCKSTEP " << ((O.checks & 64) ? 1 : 0) << "\n";
        o << "#define PG_FAST " << (O.fast ? 1 : 0) << "\n";
        // (store-time claims: not with bank / coalescing statistics, nor with PGVC_CAS=0 - api.cpp cas_on)
        if (std::getenv("PGVC_PACK_OLD"))   // (diagnostics: round 1's 16/10/26/12 event prefix)
            o << "#define PG_PACK_B0 16u\n#define PG_PACK_B1 10u\n#define PG_PACK_B2 26u\n#define PG_PACK_B3 12u\n";
        if (std::getenv("PGVC_RC_INLINE") && std::string(std::getenv("PGVC_RC_INLINE")) == "1")
            o << "#define PG_RC_INLINE __forceinline__\n";
        o << "#define PG_CAS_ON "
          << (((std::getenv("PGVC_CAS") && std::string(std::getenv("PGVC_CAS")) == "0") || (O.checks & (8 | 16))) ? 0 : 1)
          << "\n";
        o << "#define PG_DIVBAR " << (K.div_barrier ? 1 : 0) << "\n";
        o << "#define PG_OPCOUNT " << ((O.checks & 128) ? 1 : 0) << "\n";
        o << "#define PG_VCLIT " << ((O.checks & 256) ? 1 : 0) << "\n";
        o << "#define PG_WMAX " << O.wmax << "\n";
        o << "#define PG_MS " << (ms() ? O.ms : 1u) << "\n";
        o << "#define PG_NSTATS " << std::max<size_t>(1, K.sites.size()) << "\n";
        o << "#ifndef PG_VMAX\n#define PG_VMAX 1\n#endif\n";
        o << "#include \"pg_device_rt.cuh\"\n\n";
        o << "// kernel " << K.name << "\n";
        o << "struct PgK {\n  struct Frame {\n";
        for (size_t i = 0; i < K.vars.size(); i++)
            o << "    u32 v" << i << (tvar_[i] ? "[PG_MS]" : "") << ";  // " << K.vars[i].name
              << (K.vars[i].uniform ? " (uniform)" : "") << (tvar_[i] && ms() ? " (per seed)" : "") << "\n";
        for (const ArrayDecl& a : K.arrays)
            if (a.space == PRIVATE) o << "    u32 p" << a.slot << "[" << priv_size(a) << "];  // " << a.name << "\n";
        o << "    u32 pad_;\n  };\n";
        o << "  static __device__ __forceinline__ void init(Frame& F, const PgC& C, PgT& t) {\n";
        for (size_t i = 0; i < K.vars.size(); i++) {
            if (K.vars[i].scalar)
                o << "    F.v" << i << " = pg_m((u32)pg_sL.scal[" << K.vars[i].scalar_index << "]);\n";
            else if (ms() && tvar_[i])
                o << "    PG_S_LOOP F.v" << i << "[_s] = 0u;\n";
            else
                o << "    F.v" << i << " = 0u;\n";
        }
        o << "  }\n";
        // per-array claim / check dispatch for the write log (array kind fixed at code-generation time)
        o << "  static __device__ __forceinline__ void claim_one(const PgC& C, const PgT& t, u32 cell) {\n";
        o << "    const u32 flat = cell & 0xFFFFFFu;\n    switch (cell >> 24) {\n";
        for (size_t a = 0; a < K.arrays.size(); a++) {
            const ArrayDecl& A = K.arrays[a];
            if (!A.written || A.space == PRIVATE) continue;
            o << "      case " << a << ": pg_claim_" << (A.space == SHARED ? "sh" : "gt") << "<" << a
              << ">(C, t, flat); break;\n";
        }
        o << "      default: break;\n    }\n  }\n";
        o << "  static __device__ __forceinline__ void check_one(const PgC& C, PgT& t, PgCold& c, u32 cell, "
             "pg_lv_t val, u32 site) {\n";
        o << "    const u32 flat = cell & 0xFFFFFFu;\n    switch (cell >> 24) {\n";
        for (size_t a = 0; a < K.arrays.size(); a++) {
            const ArrayDecl& A = K.arrays[a];
            if (!A.written || A.space == PRIVATE) continue;
            o << "      case " << a << ": pg_check_" << (A.space == SHARED ? "sh" : "gt") << (ms() && !O.fast ? "_ms" : "")
              << "<" << a << ", "
              << (reader_tracked((int)a) ? "true" : "false") << ">(C, t, c, flat, val, site); break;\n";
        }
        o << "      default: break;\n    }\n  }\n";
        // optimistic pass: reader check of a logged cell after the round's barrier
        // (only arrays with tracked readers are logged: one such array needs no dispatch)
        o << "  static __device__ __forceinline__ void fcheck_one(const PgC& C, PgT& t, u32 cell) {\n";
        o << "    const u32 flat = cell & 0xFFFFFFu;\n";
        {
            std::vector<size_t> fa;
            for (size_t a = 0; a < K.arrays.size(); a++) {
                const ArrayDecl& A = K.arrays[a];
                if (A.written && A.space != PRIVATE && O.fast && rda_[a]) fa.push_back(a);
            }
            auto call = [&](size_t a) {
                return std::string("pg_fcheck_") + (K.arrays[a].space == SHARED ? "sh" : "gt") + "<" +
                       std::to_string(a) + ">(C, t, flat);";
            };
            if (fa.size() == 1) {
                o << "    " << call(fa[0]) << "\n";
            } else {
                o << "    switch (cell >> 24) {\n";
                for (size_t a : fa) o << "      case " << a << ": " << call(a) << " break;\n";
                o << "      default: break;\n    }\n";
            }
        }
        o << "  }\n";
        // site id of the barrier a seg() return value (resume point k >= 1) stands for (X18 records)
        o << "  static __device__ __forceinline__ u32 sync_site(u32 k) {\n    switch (k) {\n";
        for (size_t k = 0; k < seg_sites.size(); k++)
            o << "      case " << (k + 1) << "u: return " << seg_sites[k] << "u;\n";
        o << "      default: return PG_NEVER;\n    }\n  }\n";
        o << "  static __device__ __forceinline__ u32 seg(Frame& F, PgC& C, PgT& t, PgCold& c, u64* ss, u32 resume) {\n";
        o << "    switch (resume) {\n      case 0u: goto R0;\n";
        for (int k = 1; k <= seg_nsync; k++) o << "      case " << k << "u: goto R" << k << ";\n";
        o << "      default: return PG_END;\n    }\n";
        o << "R0:;\n" << seg_body;
        o << "  }\n";
        o << "  static __device__ __forceinline__ void run(Frame& F, PgC& C, PgT& t, PgCold& c, u64* ss, u32& ar) {\n";
        o << run_body;
        o << "  }\n};\n\n";
        o << "#ifndef PG_CTA_MAX\n#define PG_CTA_MAX 1024\n#define PG_MIN_BLOCKS 1\n#endif\n";
        o << "extern \"C\" __global__ void __launch_bounds__(PG_CTA_MAX, PG_MIN_BLOCKS) pgk_eval(const PgParams P) "
             "{ pg_main<PgK>(P); }\n";
        return o.str();
    }
};

}  // namespace

bool seed_oblivious(const Kernel& k, std::vector<bool>* tainted) {
    Taint T;
    T.tv.assign(k.vars.size(), false);
    for (const ArrayDecl& a : k.arrays)
        if (a.space == PRIVATE) T.ok = false;
    while (T.prop(k.body)) {
    }
    T.check(k.body);
    if (tainted) *tainted = T.tv;
    return T.ok;
}

static bool is_bid_x(const Node* n) {
    while (n && n->kind == NK::Cast && n->kids.size() == 1) n = n->kids[0];
    return n && n->kind == NK::Builtin && n->ref == 3;
}
static bool stores_bid_private(const Kernel& k, const Stmt* s) {
    if (!s) return true;
    if (s->kind == SK::Store && s->arr >= 0 && k.arrays[(size_t)s->arr].space == GLOBAL)
        if (s->index.size() != 1 || !is_bid_x(s->index[0])) return false;
    for (const Stmt* c : s->seq)
        if (!stores_bid_private(k, c)) return false;
    return stores_bid_private(k, s->body) && stores_bid_private(k, s->other) && stores_bid_private(k, s->init) &&
           stores_bid_private(k, s->step);
}
bool block_private_outputs(const Kernel& k) {
    for (const ArrayDecl& a : k.arrays)
        if (a.space == GLOBAL && a.written && a.read) return false;
    return stores_bid_private(k, k.body);
}

static const Node* strip_casts(const Node* n) {
    while (n && n->kind == NK::Cast && n->kids.size() == 1) n = n->kids[0];
    return n;
}
static bool is_tid_x(const Node* n) {
    n = strip_casts(n);
    return n && n->kind == NK::Builtin && n->ref == 0;
}
static void count_assigns(const Stmt* s, std::vector<int>& n) {
    if (!s) return;
    if (s->kind == SK::Assign && s->var >= 0) n[(size_t)s->var]++;
    for (const Stmt* c : s->seq) count_assigns(c, n);
    count_assigns(s->body, n);
    count_assigns(s->other, n);
    count_assigns(s->init, n);
    count_assigns(s->step, n);
}
static bool node_mentions(const Node* e, int v) {
    if (!e) return false;
    if (e->kind == NK::Var && e->ref == v) return true;
    for (const Node* c : e->kids)
        if (node_mentions(c, v)) return true;
    return false;
}
static bool stmt_mentions(const Stmt* s, int v) {
    if (!s) return false;
    if (s->kind == SK::Assign && s->var == v) return true;
    if (node_mentions(s->value, v) || node_mentions(s->cond, v)) return true;
    for (const Node* i : s->index)
        if (node_mentions(i, v)) return true;
    for (const Stmt* c : s->seq)
        if (stmt_mentions(c, v)) return true;
    return stmt_mentions(s->body, v) || stmt_mentions(s->other, v) || stmt_mentions(s->init, v) ||
           stmt_mentions(s->step, v);
}
struct TpCtx {
    const Kernel& k;
    std::vector<int> nassign;
    std::vector<bool> alias;   // top-level variables that hold tid.x wherever they are used
    bool tid_value(const Node* v) const {
        v = strip_casts(v);
        return is_tid_x(v) || (v && v->kind == NK::Var && v->ref >= 0 && alias[(size_t)v->ref]);
    }
};
// Store sites: index tid.x, a top-level alias, or the hidden copy a compound assignment
// `s[t] op= e` makes of its index right before the store (X21: [h = t; s[h] = s[h] op e])
static void tp_stores(const TpCtx& x, const Stmt* s, std::vector<bool>& tp) {
    if (!s) return;
    for (size_t p = 0; p < s->seq.size(); p++) {
        const Stmt* c = s->seq[p];
        if (c && c->kind == SK::Store && c->arr >= 0 && c->index.size() == 1) {
            const Node* ix = strip_casts(c->index[0]);
            if (!x.tid_value(ix) && ix && ix->kind == NK::Var && ix->ref >= 0 && p > 0) {
                const Stmt* d = s->seq[p - 1];
                const int h = ix->ref;
                if (d && d->kind == SK::Assign && d->var == h && x.nassign[(size_t)h] == 1 && x.tid_value(d->value))
                    continue;   // (the compound pattern: the store is fine)
            }
        }
        tp_stores(x, c, tp);
    }
    if (s->kind == SK::Store && s->arr >= 0) {
        if (!(s->index.size() == 1 && x.tid_value(s->index[0]))) tp[(size_t)s->arr] = false;
    }
    tp_stores(x, s->body, tp);
    tp_stores(x, s->other, tp);
    tp_stores(x, s->init, tp);
    tp_stores(x, s->step, tp);
}
static TpCtx tp_ctx(const Kernel& k);
std::vector<bool> tid_alias_vars(const Kernel& k) {
    TpCtx x = tp_ctx(k);
    // plus the hidden copies compound stores make of their index (X21): assigned once, right
    // before the store that reads and writes through them
    std::vector<bool> out = x.alias;
    struct W {
        const TpCtx& x;
        std::vector<bool>& out;
        void go(const Stmt* s) {
            if (!s) return;
            if (s->kind == SK::Assign && s->var >= 0 && x.k.vars[(size_t)s->var].hidden &&
                x.nassign[(size_t)s->var] == 1 && x.tid_value(s->value))
                out[(size_t)s->var] = true;
            for (const Stmt* c : s->seq) go(c);
            go(s->body);
            go(s->other);
            go(s->init);
            go(s->step);
        }
    } w{x, out};
    w.go(k.body);
    return out;
}
static TpCtx tp_ctx(const Kernel& k) {
    TpCtx x{k, std::vector<int>(k.vars.size(), 0), std::vector<bool>(k.vars.size(), false)};
    count_assigns(k.body, x.nassign);
    // top-level aliases: the variable's only assignment is a top-level `v = tid.x` (or `= u`,
    // u an alias defined earlier) and no earlier top-level statement mentions v (before it,
    // v holds its initial 0, X21)
    std::vector<const Stmt*> top;
    if (k.body && k.body->kind == SK::Seq) top.assign(k.body->seq.begin(), k.body->seq.end());
    else if (k.body) top.push_back(k.body);
    for (size_t i = 0; i < top.size(); i++) {
        const Stmt* st = top[i];
        if (!st || st->kind != SK::Assign || st->var < 0) continue;
        const int v = st->var;
        if (k.vars[(size_t)v].scalar || x.nassign[(size_t)v] != 1 || !x.tid_value(st->value)) continue;
        bool early = false;
        for (size_t j = 0; j < i && !early; j++) early = stmt_mentions(top[j], v);
        if (!early) x.alias[(size_t)v] = true;
    }
    return x;
}
std::vector<bool> thread_private_stores(const Kernel& k) {
    TpCtx x = tp_ctx(k);
    std::vector<bool> tp(k.arrays.size(), false);
    for (size_t a = 0; a < k.arrays.size(); a++)
        tp[a] = k.arrays[a].space == SHARED && k.arrays[a].dims.size() == 1 && k.arrays[a].written;
    tp_stores(x, k.body, tp);
    return tp;
}

std::string generate_cuda(const Kernel& k, const CodegenOptions& opt) {
    Gen g(k, opt);
    return g.run();
}

}  // namespace pgf
