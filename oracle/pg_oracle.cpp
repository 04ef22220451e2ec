/*
 * pg_oracle.cpp — the CPU ORACLE for bounded instantiation of PUGpara's
 * verification conditions.  TEST INFRASTRUCTURE ONLY: nothing on the product
 * path (paper_conf_ipps_lig12_b200/, libpgvc.so) may include, link or call
 * this file; only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline
 * leg use it (through oracle/__init__.py).  It shares no code with the CUDA
 * path: its own lexer, parser, evaluator and PRF.
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, cited as Lnnn):
 *   * concrete execution of a kernel under barrier-interval ("round")
 *     semantics, L150-L152 and L658-L662 (§II, §IV.C);
 *   * threads of one block run in NATURAL ORDER inside a round, L384-L389
 *     (§III "Serializing Concurrent Executions"); blocks run in linear bid
 *     order (they never synchronise, L107-L109);
 *   * a read sees the round-start value of the cell unless the reading thread
 *     wrote it earlier in the same round (reading X3); writes are
 *     committed at the barrier, the min-tid writer winning a WW conflict (X4);
 *   * the comparative assertion  i_s = i_t => o_s = o_t  of L438-L444 and
 *     L652-L657, instantiated for every launch and seed of the bounded space;
 *   * the race premise "at most one thread satisfies p" (L516-L520) and "no
 *     conflicts within a BI" (L660-L662) checked as WW / RW / XB races;
 *   * bank-conflict and coalescing conditions (L21-L24, L146-L150, L155) under
 *     DESIGN.md reading X9;
 *   * optional VC-literal mode: for every read, enumerate every thread s of the
 *     block and every earlier round and evaluate "s wrote this cell" literally
 *     (the fresh-writer instantiation of Fig. 2, and the nested ite
 *     of L709-L712); the result must equal the ownership-derived writer.
 *
 * Every place where the paper is silent is decided by a DESIGN.md reading
 * (X1..X21); the reading is named at the line that implements it.
 * The oracle is deliberately plain: maps, vectors, a recursive expression
 * evaluator, one thread at a time.  It is slow by design.
 */
#include <cstdint>
#include <cstdio>
#include <cstring>
#include <cctype>
#include <string>
#include <vector>
#include <map>
#include <set>
#include <algorithm>
#include <stdexcept>
#include <functional>
#include <memory>
#include <array>
#include <tuple>

namespace orc {

/* ------------------------------------------------------------------ PRF (X8) */
/* SplitMix64 (Steele/Lea/Flood; Vigna's reference constants).              */
static uint64_t sm64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ULL;
    uint64_t z = x;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}
/* RAND32(seed, tag, idx) = low32(sm(sm(seed) ^ (tag << 48) ^ idx))  (X8)     */
static uint32_t rand32(uint64_t seed, uint64_t tag, uint64_t idx) {
    return (uint32_t)sm64(sm64(seed) ^ (tag << 48) ^ idx);
}

struct Error : std::runtime_error {
    int code;
    Error(int c, const std::string& m) : std::runtime_error(m), code(c) {}
};
enum { E_ARG = -1, E_PARSE = -2, E_TYPE = -3, E_LIMIT = -4 };

static std::string at(int line, int col) {
    return std::to_string(line) + ":" + std::to_string(col) + ": ";
}

/* ------------------------------------------------------------------ lexer  */
enum { TK_EOF, TK_ID, TK_NUM, TK_OP };
struct Tok {
    int k = TK_EOF;
    std::string s;
    uint64_t v = 0;
    bool uns = false;
    bool hex = false;
    int line = 0, col = 0;
};

static std::vector<Tok> lex(const std::string& src) {
    std::vector<Tok> out;
    int line = 1, col = 1;
    size_t i = 0;
    auto adv = [&](size_t n) {
        for (size_t k = 0; k < n && i < src.size(); k++) {
            if (src[i] == '\n') { line++; col = 1; } else col++;
            i++;
        }
    };
    static const char* ops3[] = {"<<=", ">>=", nullptr};
    static const char* ops2[] = {"<<", ">>", "<=", ">=", "==", "!=", "&&", "||", "++", "--",
                                 "+=", "-=", "*=", "/=", "%=", "&=", "|=", "^=", nullptr};
    while (i < src.size()) {
        char c = src[i];
        if (isspace((unsigned char)c)) { adv(1); continue; }
        if (c == '/' && i + 1 < src.size() && src[i + 1] == '/') {
            while (i < src.size() && src[i] != '\n') adv(1);
            continue;
        }
        if (c == '/' && i + 1 < src.size() && src[i + 1] == '*') {
            int l0 = line, c0 = col;
            adv(2);
            while (i + 1 < src.size() && !(src[i] == '*' && src[i + 1] == '/')) adv(1);
            if (i + 1 >= src.size()) throw Error(E_PARSE, at(l0, c0) + "unterminated comment");
            adv(2);
            continue;
        }
        Tok t;
        t.line = line; t.col = col;
        if (isalpha((unsigned char)c) || c == '_') {
            size_t j = i;
            while (j < src.size() && (isalnum((unsigned char)src[j]) || src[j] == '_')) j++;
            t.k = TK_ID; t.s = src.substr(i, j - i);
            adv(j - i);
            out.push_back(t);
            continue;
        }
        if (isdigit((unsigned char)c)) {
            size_t j = i;
            uint64_t v = 0;
            bool hex = false;
            if (c == '0' && j + 1 < src.size() && (src[j + 1] == 'x' || src[j + 1] == 'X')) {
                hex = true;
                j += 2;
                size_t d0 = j;
                while (j < src.size() && isxdigit((unsigned char)src[j])) {
                    char h = (char)tolower(src[j]);
                    v = v * 16 + (uint64_t)(isdigit((unsigned char)h) ? h - '0' : h - 'a' + 10);
                    if (v > 0xFFFFFFFFULL) throw Error(E_PARSE, at(line, col) + "integer literal too large");
                    j++;
                }
                if (j == d0) throw Error(E_PARSE, at(line, col) + "bad hex literal");
            } else {
                while (j < src.size() && isdigit((unsigned char)src[j])) {
                    v = v * 10 + (uint64_t)(src[j] - '0');
                    if (v > 0xFFFFFFFFULL) throw Error(E_PARSE, at(line, col) + "integer literal too large");
                    j++;
                }
            }
            bool uns = false;
            while (j < src.size() && (src[j] == 'u' || src[j] == 'U' || src[j] == 'l' || src[j] == 'L')) {
                if (src[j] == 'u' || src[j] == 'U') uns = true;
                j++;
            }
            if (j < src.size() && (isalnum((unsigned char)src[j]) || src[j] == '_'))
                throw Error(E_PARSE, at(line, col) + "bad integer literal");
            t.k = TK_NUM; t.v = v; t.uns = uns; t.hex = hex;
            t.s = src.substr(i, j - i);
            adv(j - i);
            out.push_back(t);
            continue;
        }
        bool matched = false;
        for (int n = 3; n >= 2 && !matched; n--) {
            const char** tab = (n == 3) ? ops3 : ops2;
            for (int q = 0; tab[q]; q++) {
                if (src.compare(i, (size_t)n, tab[q]) == 0) {
                    t.k = TK_OP; t.s = tab[q];
                    adv((size_t)n);
                    matched = true;
                    break;
                }
            }
        }
        if (!matched) {
            if (strchr("+-*/%<>=!~&|^?:;,.()[]{}", c) == nullptr)
                throw Error(E_PARSE, at(line, col) + std::string("unexpected character '") + c + "'");
            t.k = TK_OP; t.s = std::string(1, c);
            adv(1);
        }
        out.push_back(t);
    }
    Tok e;
    e.k = TK_EOF; e.line = line; e.col = col;
    out.push_back(e);
    return out;
}

/* ------------------------------------------------------------------ AST    */
enum { TY_INT = 0, TY_UNS = 1 };
enum {
    EX_NUM, EX_VAR, EX_BUILTIN, EX_LOAD, EX_NEG, EX_BNOT, EX_LNOT, EX_BIN,
    EX_LAND, EX_LOR, EX_COND, EX_MIN, EX_MAX, EX_CAST
};
enum {
    B_ADD, B_SUB, B_MUL, B_DIV, B_REM, B_SHL, B_SHR, B_AND, B_OR, B_XOR,
    B_LT, B_LE, B_GT, B_GE, B_EQ, B_NE
};
/* builtins (L114-L116): tid.xyz, bid.xyz, bdim.xyz, gdim.xyz */
enum { BI_TID = 0, BI_BID = 3, BI_BDIM = 6, BI_GDIM = 9 };

struct Expr {
    int k = EX_NUM;
    int ty = TY_INT;     /* result type */
    int opty = TY_INT;   /* type the operation is performed in (C usual conversions) */
    uint32_t num = 0;
    int var = -1, bi = -1, arr = -1, site = -1, op = -1;
    std::vector<Expr*> idx;
    Expr *a = nullptr, *b = nullptr, *c = nullptr;
    int line = 0, col = 0;
};

enum { SP_GLOBAL = 0, SP_SHARED = 1, SP_PRIVATE = 2 };
enum { M_IN = 0, M_OUT = 1, M_INOUT = 2 };

struct Arr {
    std::string name;
    int space = SP_GLOBAL;
    int ety = TY_INT;
    int mode = M_IN;
    std::vector<Expr*> dims;   /* global: one size expr; shared: dims; private: constant dims */
    int local_index = 0;       /* index among arrays of its space, in declaration order */
};

struct Var {
    std::string name;
    int ty = TY_INT;
};

enum {
    ST_BLOCK, ST_ASSIGN, ST_STORE, ST_PDECL, ST_IF, ST_LOOP, ST_SYNC, ST_RETURN,
    ST_BREAK, ST_CONTINUE, ST_NOP
};
struct Stmt {
    int k = ST_NOP;
    std::vector<Stmt*> body;
    int var = -1;
    Expr* e = nullptr;            /* assigned value / store value / if-cond / loop-cond */
    int arr = -1;
    std::vector<Expr*> idx;
    int site = -1;
    Stmt *then_s = nullptr, *else_s = nullptr;
    Stmt *init = nullptr, *step = nullptr, *lbody = nullptr;
    int loop_id = -1;
    int line = 0, col = 0;
};

struct Kernel {
    std::string name;
    std::vector<Var> vars;
    std::vector<Arr> arrs;
    std::vector<int> scalar_vars;   /* var index of each scalar parameter, in order */
    Stmt* body = nullptr;
    int n_sites = 0;
    int n_loops = 0;
    std::vector<std::vector<int>> site_loops;  /* enclosing loop ids of each site, outermost first */
    std::vector<int> site_arr;                 /* array of an access site, -1 for sync sites */
    std::vector<std::unique_ptr<Expr>> expr_pool;
    std::vector<std::unique_ptr<Stmt>> stmt_pool;
};

/* ------------------------------------------------------------------ parser */
struct Parser {
    std::vector<Tok> t;
    size_t p = 0;
    Kernel* K;
    std::vector<std::map<std::string, int>> scopes;      /* name -> var index */
    std::map<std::string, int> arr_by_name;              /* arrays: globals, shared, privates are all unique-named */
    std::vector<int> loop_stack;
    int n_hidden = 0;

    Parser(const std::string& src, Kernel* k) : t(lex(src)), K(k) {}

    const Tok& cur() { return t[p]; }
    bool is_op(const char* s) { return cur().k == TK_OP && cur().s == s; }
    bool is_id(const char* s) { return cur().k == TK_ID && cur().s == s; }
    [[noreturn]] void fail(const std::string& m) { throw Error(E_PARSE, at(cur().line, cur().col) + m); }
    [[noreturn]] void tfail(int line, int col, const std::string& m) { throw Error(E_TYPE, at(line, col) + m); }
    void expect(const char* s) {
        if (!is_op(s)) fail(std::string("expected '") + s + "'");
        p++;
    }
    std::string ident() {
        if (cur().k != TK_ID) fail("expected identifier");
        return t[p++].s;
    }
    Expr* ne(int k, const Tok& at_tok) {
        K->expr_pool.emplace_back(new Expr());
        Expr* e = K->expr_pool.back().get();
        e->k = k; e->line = at_tok.line; e->col = at_tok.col;
        return e;
    }
    Stmt* ns(int k, const Tok& at_tok) {
        K->stmt_pool.emplace_back(new Stmt());
        Stmt* s = K->stmt_pool.back().get();
        s->k = k; s->line = at_tok.line; s->col = at_tok.col;
        return s;
    }
    int new_site(int arr) {
        K->site_loops.push_back(loop_stack);
        K->site_arr.push_back(arr);
        return K->n_sites++;
    }
    bool is_type_kw() { return is_id("int") || is_id("unsigned"); }
    int parse_type() {
        if (is_id("int")) { p++; return TY_INT; }
        if (is_id("unsigned")) { p++; if (is_id("int")) p++; return TY_UNS; }
        fail("expected type");
    }
    static bool reserved(const std::string& s) {
        static const char* kw[] = {"int", "unsigned", "kernel", "global", "shared", "__shared__", "if", "else",
                                   "for", "while", "sync", "__syncthreads", "return", "break", "continue",
                                   "in", "out", "inout", "min", "max", "tid", "bid", "bdim", "gdim",
                                   "threadIdx", "blockIdx", "blockDim", "gridDim", nullptr};
        for (int i = 0; kw[i]; i++) if (s == kw[i]) return true;
        return false;
    }
    int declare_var(const std::string& name, int ty, const Tok& tk) {
        if (reserved(name)) tfail(tk.line, tk.col, "reserved name '" + name + "'");
        if (scopes.back().count(name) || arr_by_name.count(name))
            tfail(tk.line, tk.col, "redeclaration of '" + name + "'");
        Var v; v.name = name; v.ty = ty;
        K->vars.push_back(v);
        scopes.back()[name] = (int)K->vars.size() - 1;
        return (int)K->vars.size() - 1;
    }
    int hidden_var(int ty) {
        Var v; v.name = "$t" + std::to_string(n_hidden++); v.ty = ty;
        K->vars.push_back(v);
        return (int)K->vars.size() - 1;
    }
    int lookup_var(const std::string& name) {
        for (int i = (int)scopes.size() - 1; i >= 0; i--) {
            auto it = scopes[(size_t)i].find(name);
            if (it != scopes[(size_t)i].end()) return it->second;
        }
        return -1;
    }

    /* C usual arithmetic conversions on {int, unsigned} */
    static int conv(int a, int b) { return (a == TY_UNS || b == TY_UNS) ? TY_UNS : TY_INT; }

    /* --- expressions, C precedence --- */
    Expr* expr() { return cond_expr(); }
    Expr* cond_expr() {
        Expr* c = lor();
        if (is_op("?")) {
            Tok tk = cur(); p++;
            Expr* a = expr();
            expect(":");
            Expr* b = cond_expr();
            Expr* e = ne(EX_COND, tk);
            e->a = c; e->b = a; e->c = b;
            e->ty = e->opty = conv(a->ty, b->ty);
            return e;
        }
        return c;
    }
    Expr* lor() {
        Expr* l = land();
        while (is_op("||")) {
            Tok tk = cur(); p++;
            Expr* r = land();
            Expr* e = ne(EX_LOR, tk); e->a = l; e->b = r; e->ty = TY_INT;
            l = e;
        }
        return l;
    }
    Expr* land() {
        Expr* l = bor();
        while (is_op("&&")) {
            Tok tk = cur(); p++;
            Expr* r = bor();
            Expr* e = ne(EX_LAND, tk); e->a = l; e->b = r; e->ty = TY_INT;
            l = e;
        }
        return l;
    }
    Expr* mkbin(int op, Expr* l, Expr* r, const Tok& tk) {
        Expr* e = ne(EX_BIN, tk);
        e->op = op; e->a = l; e->b = r;
        if (op == B_SHL || op == B_SHR) { e->opty = l->ty; e->ty = l->ty; }
        else if (op >= B_LT) { e->opty = conv(l->ty, r->ty); e->ty = TY_INT; }
        else { e->opty = conv(l->ty, r->ty); e->ty = e->opty; }
        return e;
    }
    Expr* bor() {
        Expr* l = bxor();
        while (is_op("|")) { Tok tk = cur(); p++; l = mkbin(B_OR, l, bxor(), tk); }
        return l;
    }
    Expr* bxor() {
        Expr* l = band();
        while (is_op("^")) { Tok tk = cur(); p++; l = mkbin(B_XOR, l, band(), tk); }
        return l;
    }
    Expr* band() {
        Expr* l = equality();
        while (is_op("&")) { Tok tk = cur(); p++; l = mkbin(B_AND, l, equality(), tk); }
        return l;
    }
    Expr* equality() {
        Expr* l = relational();
        for (;;) {
            if (is_op("==")) { Tok tk = cur(); p++; l = mkbin(B_EQ, l, relational(), tk); }
            else if (is_op("!=")) { Tok tk = cur(); p++; l = mkbin(B_NE, l, relational(), tk); }
            else return l;
        }
    }
    Expr* relational() {
        Expr* l = shift();
        for (;;) {
            int op = -1;
            if (is_op("<")) op = B_LT; else if (is_op("<=")) op = B_LE;
            else if (is_op(">")) op = B_GT; else if (is_op(">=")) op = B_GE;
            if (op < 0) return l;
            Tok tk = cur(); p++;
            l = mkbin(op, l, shift(), tk);
        }
    }
    Expr* shift() {
        Expr* l = additive();
        for (;;) {
            if (is_op("<<")) { Tok tk = cur(); p++; l = mkbin(B_SHL, l, additive(), tk); }
            else if (is_op(">>")) { Tok tk = cur(); p++; l = mkbin(B_SHR, l, additive(), tk); }
            else return l;
        }
    }
    Expr* additive() {
        Expr* l = mult();
        for (;;) {
            if (is_op("+")) { Tok tk = cur(); p++; l = mkbin(B_ADD, l, mult(), tk); }
            else if (is_op("-")) { Tok tk = cur(); p++; l = mkbin(B_SUB, l, mult(), tk); }
            else return l;
        }
    }
    Expr* mult() {
        Expr* l = unary();
        for (;;) {
            if (is_op("*")) { Tok tk = cur(); p++; l = mkbin(B_MUL, l, unary(), tk); }
            else if (is_op("/")) { Tok tk = cur(); p++; l = mkbin(B_DIV, l, unary(), tk); }
            else if (is_op("%")) { Tok tk = cur(); p++; l = mkbin(B_REM, l, unary(), tk); }
            else return l;
        }
    }
    Expr* unary() {
        Tok tk = cur();
        if (is_op("-")) { p++; Expr* a = unary(); Expr* e = ne(EX_NEG, tk); e->a = a; e->ty = a->ty; return e; }
        if (is_op("+")) { p++; return unary(); }
        if (is_op("~")) { p++; Expr* a = unary(); Expr* e = ne(EX_BNOT, tk); e->a = a; e->ty = a->ty; return e; }
        if (is_op("!")) { p++; Expr* a = unary(); Expr* e = ne(EX_LNOT, tk); e->a = a; e->ty = TY_INT; return e; }
        if (is_op("(") && t[p + 1].k == TK_ID && (t[p + 1].s == "int" || t[p + 1].s == "unsigned")) {
            p++;
            int ty = parse_type();
            expect(")");
            Expr* a = unary();
            Expr* e = ne(EX_CAST, tk); e->a = a; e->ty = ty;
            return e;
        }
        return primary();
    }
    int builtin_base(const std::string& s) {
        if (s == "tid" || s == "threadIdx") return BI_TID;
        if (s == "bid" || s == "blockIdx") return BI_BID;
        if (s == "bdim" || s == "blockDim") return BI_BDIM;
        if (s == "gdim" || s == "gridDim") return BI_GDIM;
        return -1;
    }
    /* array element reference: NAME [e] [e]... ; sites allocated by caller */
    void parse_indices(int arr, std::vector<Expr*>& idx) {
        const Arr& A = K->arrs[(size_t)arr];
        size_t nd = A.space == SP_GLOBAL ? 1 : A.dims.size();
        for (size_t d = 0; d < nd; d++) {
            expect("[");
            idx.push_back(expr());
            expect("]");
        }
        if (is_op("[")) fail("too many indices for array '" + A.name + "'");
    }
    Expr* primary() {
        Tok tk = cur();
        if (tk.k == TK_NUM) {
            p++;
            Expr* e = ne(EX_NUM, tk);
            e->num = (uint32_t)tk.v;
            /* literal typing: int if it fits in int and has no u suffix, else unsigned */
            e->ty = (tk.uns || tk.v > 0x7FFFFFFFULL) ? TY_UNS : TY_INT;
            return e;
        }
        if (is_op("(")) {
            p++;
            Expr* e = expr();
            expect(")");
            return e;
        }
        if (tk.k == TK_ID) {
            if (tk.s == "min" || tk.s == "max") {
                p++;
                expect("(");
                Expr* a = expr();
                expect(",");
                Expr* b = expr();
                expect(")");
                Expr* e = ne(tk.s == "min" ? EX_MIN : EX_MAX, tk);
                e->a = a; e->b = b; e->ty = e->opty = conv(a->ty, b->ty);
                return e;
            }
            int bb = builtin_base(tk.s);
            if (bb >= 0) {
                p++;
                expect(".");
                std::string f = ident();
                int comp = f == "x" ? 0 : f == "y" ? 1 : f == "z" ? 2 : -1;
                if (comp < 0) fail("expected .x, .y or .z");
                Expr* e = ne(EX_BUILTIN, tk);
                e->bi = bb + comp;
                e->ty = TY_UNS;   /* CUDA's uint3 builtins are unsigned (X2) */
                return e;
            }
            p++;
            auto ai = arr_by_name.find(tk.s);
            if (ai != arr_by_name.end()) {
                Expr* e = ne(EX_LOAD, tk);
                e->arr = ai->second;
                parse_indices(e->arr, e->idx);
                e->site = new_site(e->arr);
                e->ty = K->arrs[(size_t)e->arr].ety;
                return e;
            }
            int v = lookup_var(tk.s);
            if (v < 0) tfail(tk.line, tk.col, "undeclared identifier '" + tk.s + "'");
            Expr* e = ne(EX_VAR, tk);
            e->var = v; e->ty = K->vars[(size_t)v].ty;
            return e;
        }
        fail("expected expression");
    }

    /* --- statements --- */
    Stmt* block_of(std::vector<Stmt*> v, const Tok& tk) {
        Stmt* s = ns(ST_BLOCK, tk);
        s->body = std::move(v);
        return s;
    }
    Expr* mkvar(int v, const Tok& tk) {
        Expr* e = ne(EX_VAR, tk); e->var = v; e->ty = K->vars[(size_t)v].ty; return e;
    }
    Expr* mknum(uint32_t n, const Tok& tk) {
        Expr* e = ne(EX_NUM, tk); e->num = n; e->ty = TY_INT; return e;
    }
    int compound_op(const std::string& s) {
        static const char* names[] = {"+=", "-=", "*=", "/=", "%=", "<<=", ">>=", "&=", "|=", "^="};
        static const int ops[] = {B_ADD, B_SUB, B_MUL, B_DIV, B_REM, B_SHL, B_SHR, B_AND, B_OR, B_XOR};
        for (int i = 0; i < 10; i++) if (s == names[i]) return ops[i];
        return -1;
    }
    /* simple statement: assignment / compound assignment / ++ / -- (no trailing ';') */
    Stmt* simple_stmt() {
        Tok tk = cur();
        bool pre_inc = false, pre_dec = false;
        if (is_op("++")) { pre_inc = true; p++; }
        else if (is_op("--")) { pre_dec = true; p++; }
        Tok nt = cur();
        std::string name = ident();
        auto ai = arr_by_name.find(name);
        if (ai != arr_by_name.end()) {
            int arr = ai->second;
            std::vector<Expr*> idx;
            parse_indices(arr, idx);
            int s1 = new_site(arr);
            int op = -1;
            Expr* rhs = nullptr;
            bool simple = false;
            if (pre_inc || pre_dec) { op = pre_inc ? B_ADD : B_SUB; rhs = mknum(1, tk); }
            else if (is_op("=")) { p++; simple = true; }
            else if (is_op("++") || is_op("--")) { op = is_op("++") ? B_ADD : B_SUB; p++; rhs = mknum(1, tk); }
            else if ((op = compound_op(cur().s)) >= 0 && cur().k == TK_OP) { p++; }
            else fail("expected assignment");
            if (simple) {
                Stmt* s = ns(ST_STORE, nt);
                s->arr = arr; s->idx = idx; s->site = s1;
                s->e = expr();
                return s;
            }
            /* compound: read site s1, write site s1+1 (allocated now, before the RHS) */
            int s2 = new_site(arr);
            if (!rhs) rhs = expr();
            /* evaluate each index once into hidden temporaries (X21) */
            std::vector<Stmt*> seq;
            std::vector<Expr*> tidx;
            for (Expr* ie : idx) {
                int hv = hidden_var(ie->ty);
                Stmt* as = ns(ST_ASSIGN, nt); as->var = hv; as->e = ie;
                seq.push_back(as);
                tidx.push_back(mkvar(hv, nt));
            }
            Expr* ld = ne(EX_LOAD, nt);
            ld->arr = arr; ld->idx = tidx; ld->site = s1; ld->ty = K->arrs[(size_t)arr].ety;
            Stmt* st = ns(ST_STORE, nt);
            st->arr = arr; st->idx = tidx; st->site = s2;
            st->e = mkbin(op, ld, rhs, nt);
            seq.push_back(st);
            return block_of(seq, nt);
        }
        int v = lookup_var(name);
        if (v < 0) tfail(nt.line, nt.col, "undeclared identifier '" + name + "'");
        Stmt* s = ns(ST_ASSIGN, nt);
        s->var = v;
        int op = -1;
        Expr* rhs = nullptr;
        if (pre_inc || pre_dec) { op = pre_inc ? B_ADD : B_SUB; rhs = mknum(1, tk); }
        else if (is_op("=")) { p++; s->e = expr(); return s; }
        else if (is_op("++") || is_op("--")) { op = is_op("++") ? B_ADD : B_SUB; p++; rhs = mknum(1, tk); }
        else if (cur().k == TK_OP && (op = compound_op(cur().s)) >= 0) { p++; rhs = expr(); }
        else fail("expected assignment");
        s->e = mkbin(op, mkvar(v, nt), rhs, nt);
        return s;
    }
    /* declaration: type NAME ([N])? (= e)? (, ...)*  (no trailing ';') */
    Stmt* decl_stmt() {
        Tok tk = cur();
        int ty = parse_type();
        std::vector<Stmt*> seq;
        for (;;) {
            Tok nt = cur();
            std::string name = ident();
            if (is_op("[")) {
                /* private per-thread array with constant dims (zero-initialised, X21) */
                if (reserved(name) || scopes.back().count(name) || arr_by_name.count(name) || lookup_var(name) >= 0)
                    tfail(nt.line, nt.col, "redeclaration of '" + name + "'");
                Arr A; A.name = name; A.space = SP_PRIVATE; A.ety = ty;
                int np = 0;
                for (auto& a : K->arrs) if (a.space == SP_PRIVATE) np++;
                A.local_index = np;
                while (is_op("[")) {
                    p++;
                    if (cur().k != TK_NUM) fail("private array dimension must be an integer literal");
                    A.dims.push_back(mknum((uint32_t)cur().v, cur()));
                    p++;
                    expect("]");
                }
                K->arrs.push_back(A);
                arr_by_name[name] = (int)K->arrs.size() - 1;
                Stmt* s = ns(ST_PDECL, nt);
                s->arr = (int)K->arrs.size() - 1;
                seq.push_back(s);
            } else {
                Expr* init = nullptr;
                if (is_op("=")) { p++; init = expr(); }
                int v = declare_var(name, ty, nt);   /* declared after its initialiser (C scoping) */
                Stmt* s = ns(ST_ASSIGN, nt);
                s->var = v;
                s->e = init ? init : mknum(0, nt);   /* uninitialised locals read as 0 (X21) */
                seq.push_back(s);
            }
            if (is_op(",")) { p++; continue; }
            break;
        }
        if (seq.size() == 1) return seq[0];
        return block_of(seq, tk);
    }
    Stmt* statement() {
        Tok tk = cur();
        if (is_op("{")) {
            p++;
            scopes.emplace_back();
            std::vector<Stmt*> v;
            while (!is_op("}")) {
                if (cur().k == TK_EOF) fail("unexpected end of input");
                v.push_back(statement());
            }
            p++;
            scopes.pop_back();
            return block_of(v, tk);
        }
        if (is_op(";")) { p++; return ns(ST_NOP, tk); }
        if (is_id("shared") || is_id("__shared__")) fail("shared declarations must be at the top level of the kernel body");
        if (is_type_kw()) {
            Stmt* s = decl_stmt();
            expect(";");
            return s;
        }
        if (is_id("if")) {
            p++;
            expect("(");
            Expr* c = expr();
            expect(")");
            Stmt* s = ns(ST_IF, tk);
            s->e = c;
            scopes.emplace_back(); s->then_s = statement(); scopes.pop_back();
            if (is_id("else")) { p++; scopes.emplace_back(); s->else_s = statement(); scopes.pop_back(); }
            return s;
        }
        if (is_id("for")) {
            p++;
            Stmt* s = ns(ST_LOOP, tk);
            s->loop_id = K->n_loops++;
            scopes.emplace_back();
            expect("(");
            if (!is_op(";")) s->init = is_type_kw() ? decl_stmt() : simple_stmt();
            expect(";");
            loop_stack.push_back(s->loop_id);
            if (!is_op(";")) s->e = expr();
            expect(";");
            if (!is_op(")")) s->step = simple_stmt();
            expect(")");
            scopes.emplace_back();
            s->lbody = statement();
            scopes.pop_back();
            loop_stack.pop_back();
            scopes.pop_back();
            return s;
        }
        if (is_id("while")) {
            p++;
            Stmt* s = ns(ST_LOOP, tk);
            s->loop_id = K->n_loops++;
            loop_stack.push_back(s->loop_id);
            expect("(");
            s->e = expr();
            expect(")");
            scopes.emplace_back();
            s->lbody = statement();
            scopes.pop_back();
            loop_stack.pop_back();
            return s;
        }
        if (is_id("sync") || is_id("__syncthreads")) {
            bool cu = is_id("__syncthreads");
            p++;
            if (cu) { expect("("); expect(")"); }
            expect(";");
            Stmt* s = ns(ST_SYNC, tk);
            s->site = new_site(-1);
            return s;
        }
        if (is_id("return")) { p++; expect(";"); return ns(ST_RETURN, tk); }
        if (is_id("break")) {
            p++; expect(";");
            if (loop_stack.empty()) tfail(tk.line, tk.col, "break outside a loop");
            return ns(ST_BREAK, tk);
        }
        if (is_id("continue")) {
            p++; expect(";");
            if (loop_stack.empty()) tfail(tk.line, tk.col, "continue outside a loop");
            return ns(ST_CONTINUE, tk);
        }
        Stmt* s = simple_stmt();
        expect(";");
        return s;
    }
    void kernel() {
        if (!is_id("kernel")) fail("expected 'kernel'");
        p++;
        K->name = ident();
        expect("(");
        scopes.emplace_back();
        struct PendingSize { int arr; size_t tokpos; };
        std::vector<PendingSize> pending;
        std::vector<std::string> gnames;
        if (!is_op(")")) {
            for (;;) {
                Tok tk = cur();
                if (is_id("global")) {
                    p++;
                    Arr A; A.space = SP_GLOBAL;
                    if (is_id("in")) { A.mode = M_IN; p++; }
                    else if (is_id("out")) { A.mode = M_OUT; p++; }
                    else if (is_id("inout")) { A.mode = M_INOUT; p++; }
                    else fail("expected in, out or inout");
                    A.ety = parse_type();
                    Tok nt = cur();
                    A.name = ident();
                    if (reserved(A.name) || arr_by_name.count(A.name)) tfail(nt.line, nt.col, "bad or duplicate array name");
                    expect("[");
                    /* the size expression may mention scalar parameters declared later: parse it after the list */
                    size_t start = p;
                    int depth = 1;
                    while (depth > 0) {
                        if (cur().k == TK_EOF) fail("unterminated array size");
                        if (is_op("[")) depth++;
                        if (is_op("]")) depth--;
                        p++;
                    }
                    int ng = 0;
                    for (auto& a : K->arrs) if (a.space == SP_GLOBAL) ng++;
                    A.local_index = ng;
                    K->arrs.push_back(A);
                    arr_by_name[A.name] = (int)K->arrs.size() - 1;
                    pending.push_back({(int)K->arrs.size() - 1, start});
                } else if (is_type_kw()) {
                    int ty = parse_type();
                    Tok nt = cur();
                    std::string name = ident();
                    int v = declare_var(name, ty, nt);
                    K->scalar_vars.push_back(v);
                } else fail("expected parameter");
                if (is_op(",")) { p++; continue; }
                break;
            }
        }
        expect(")");
        size_t after = p;
        for (auto& ps : pending) {
            p = ps.tokpos;
            int nsites = K->n_sites;
            Expr* e = expr();
            if (K->n_sites != nsites) tfail(t[ps.tokpos].line, t[ps.tokpos].col, "array size may not read memory");
            K->arrs[(size_t)ps.arr].dims.push_back(e);
            expect("]");
        }
        p = after;
        if (K->scalar_vars.size() > 8) fail("at most 8 scalar parameters");
        expect("{");
        std::vector<Stmt*> v;
        scopes.emplace_back();
        while (!is_op("}")) {
            if (cur().k == TK_EOF) fail("unexpected end of input");
            if (is_id("shared") || is_id("__shared__")) {
                Tok st = cur();
                p++;
                Arr A; A.space = SP_SHARED;
                A.ety = parse_type();
                Tok nt = cur();
                A.name = ident();
                if (reserved(A.name) || arr_by_name.count(A.name) || lookup_var(A.name) >= 0)
                    tfail(nt.line, nt.col, "bad or duplicate array name");
                int nsites = K->n_sites;
                while (is_op("[")) { p++; A.dims.push_back(expr()); expect("]"); }
                if (A.dims.empty()) fail("shared array needs dimensions");
                if (K->n_sites != nsites) tfail(nt.line, nt.col, "array dimension may not read memory");
                int nsh = 0;
                for (auto& a : K->arrs) if (a.space == SP_SHARED) nsh++;
                A.local_index = nsh;
                K->arrs.push_back(A);
                arr_by_name[A.name] = (int)K->arrs.size() - 1;
                expect(";");
                (void)st;
                continue;
            }
            v.push_back(statement());
        }
        p++;
        scopes.pop_back();
        scopes.pop_back();
        K->body = block_of(v, t[0]);
        if (cur().k != TK_EOF) fail("trailing input after kernel");
    }
};

/* ------------------------------------------------------------------ lowering
 * The statement tree is lowered to a flat list so that a thread can stop at a
 * barrier and resume after it (a per-thread program counter).  Expressions stay
 * trees and are evaluated recursively.                                        */
enum { IN_ASSIGN, IN_STORE, IN_PDECL, IN_JZ, IN_JMP, IN_SYNC, IN_RET, IN_LENTER, IN_LNEXT, IN_END };
struct Ins {
    int k = IN_END;
    int var = -1, arr = -1, site = -1, target = -1, loop_id = -1;
    Expr* e = nullptr;
    std::vector<Expr*> idx;
};
struct Prog {
    std::vector<Ins> ins;
};
struct Lowerer {
    Prog& P;
    struct LoopCtx { std::vector<int> breaks, conts; };
    std::vector<LoopCtx> loops;
    explicit Lowerer(Prog& p) : P(p) {}
    int emit(Ins i) { P.ins.push_back(i); return (int)P.ins.size() - 1; }
    void lower(Stmt* s) {
        switch (s->k) {
        case ST_BLOCK: for (Stmt* c : s->body) lower(c); break;
        case ST_NOP: break;
        case ST_ASSIGN: { Ins i; i.k = IN_ASSIGN; i.var = s->var; i.e = s->e; emit(i); break; }
        case ST_STORE: { Ins i; i.k = IN_STORE; i.arr = s->arr; i.idx = s->idx; i.e = s->e; i.site = s->site; emit(i); break; }
        case ST_PDECL: { Ins i; i.k = IN_PDECL; i.arr = s->arr; emit(i); break; }
        case ST_SYNC: { Ins i; i.k = IN_SYNC; i.site = s->site; emit(i); break; }
        case ST_RETURN: { Ins i; i.k = IN_RET; emit(i); break; }
        case ST_BREAK: { Ins i; i.k = IN_JMP; loops.back().breaks.push_back(emit(i)); break; }
        case ST_CONTINUE: { Ins i; i.k = IN_JMP; loops.back().conts.push_back(emit(i)); break; }
        case ST_IF: {
            Ins jz; jz.k = IN_JZ; jz.e = s->e;
            int a = emit(jz);
            lower(s->then_s);
            if (s->else_s) {
                Ins j; j.k = IN_JMP;
                int b = emit(j);
                P.ins[(size_t)a].target = (int)P.ins.size();
                lower(s->else_s);
                P.ins[(size_t)b].target = (int)P.ins.size();
            } else {
                P.ins[(size_t)a].target = (int)P.ins.size();
            }
            break;
        }
        case ST_LOOP: {
            /* init; LENTER; head: JZ cond exit; body; step_label: step; LNEXT; JMP head; exit: */
            if (s->init) lower(s->init);
            Ins le; le.k = IN_LENTER; le.loop_id = s->loop_id;
            emit(le);
            int head = (int)P.ins.size();
            int jzpos = -1;
            if (s->e) { Ins jz; jz.k = IN_JZ; jz.e = s->e; jzpos = emit(jz); }
            loops.emplace_back();
            lower(s->lbody);
            int step_label = (int)P.ins.size();
            if (s->step) lower(s->step);
            Ins ln; ln.k = IN_LNEXT; ln.loop_id = s->loop_id;
            emit(ln);
            Ins j; j.k = IN_JMP; j.target = head;
            emit(j);
            int exit_label = (int)P.ins.size();
            if (jzpos >= 0) P.ins[(size_t)jzpos].target = exit_label;
            for (int b : loops.back().breaks) P.ins[(size_t)b].target = exit_label;
            for (int c : loops.back().conts) P.ins[(size_t)c].target = step_label;
            loops.pop_back();
            break;
        }
        default: throw Error(E_ARG, "internal: bad statement");
        }
    }
};

/* ------------------------------------------------------------------ public types */
struct Launch {
    uint32_t gdim[3], bdim[3];
    int32_t scalar[8];
    uint32_t n_scalar;
};

enum {
    K_BARRIER_DIV = 0, K_OOB = 1, K_RACE_WW = 2, K_RACE_RW = 3, K_RACE_XB = 4,
    K_MISMATCH = 5, K_BANK = 6, K_UNCOALESCED = 7, K_UNINIT = 8, K_LIMIT = 9, N_KINDS = 10
};
enum { CHK_EQUIV = 1, CHK_RACE = 2, CHK_OOB = 4, CHK_BANK = 8, CHK_COALESCE = 16 };
enum { IN_RAND32 = 0, IN_BITS01 = 1, IN_RANGE = 2 };
enum { MODE_EQUIV = 0, MODE_RACES = 1, MODE_BANKS = 2 };
static const uint32_t NONE32 = 0xFFFFFFFFu;
static const uint32_t ROUND_END = 0xFFFFu;     /* round field of MISMATCH / XB records */
static const uint32_t ROUND_LIMIT = 0xFFFEu;   /* rounds 0..0xFFFD run; threads still live then stop (LIMIT) */

/* One record per slot (instance, kernel, kind): the minimum event by
 * (round, array, addr, tid_a, tid_b, site, val_a, val_b) plus the event count
 * (X16).                                                                     */
struct Ev {
    uint32_t f[8];   /* round, array, addr, tid_a, tid_b, site, val_a, val_b */
};
struct Slot {
    bool has = false;
    uint64_t count = 0;
    Ev best{};
    void add(const Ev& e, uint64_t n = 1) {
        count += n;
        if (!has || std::lexicographical_compare(e.f, e.f + 8, best.f, best.f + 8)) { best = e; has = true; }
    }
};

struct SlotSet {
    Slot s[N_KINDS];
};

struct Rec {
    uint64_t key, count;
    uint32_t kind, launch, seed_idx, kernel, round, site, array, addr, tid_a, tid_b, val_a, val_b;
};

/* X16: key = launch(19) | seed_idx(21) | kernel(4) | kind(4) | round(16) */
static uint64_t make_key(uint32_t launch, uint32_t seed_idx, uint32_t kernel, uint32_t kind, uint32_t round) {
    return ((uint64_t)launch << 45) | ((uint64_t)seed_idx << 24) | ((uint64_t)kernel << 20) |
           ((uint64_t)kind << 16) | (uint64_t)(round & 0xFFFFu);
}

/* ------------------------------------------------------------------ executor */
struct Cell {
    int arr;
    uint32_t addr;
    bool operator<(const Cell& o) const { return arr != o.arr ? arr < o.arr : addr < o.addr; }
    bool operator==(const Cell& o) const { return arr == o.arr && addr == o.addr; }
};

struct WEntry {
    Cell c;
    uint32_t val;
    int site;
};

struct Thread {
    uint32_t tid[3];
    uint32_t tlin = 0;
    uint32_t gtid = 0;
    int pc = 0;
    bool exited = false;
    bool at_bar = false;
    int bar_site = -1;
    std::vector<uint32_t> vars;
    std::vector<std::vector<uint32_t>> parr;
    std::vector<uint32_t> loopctr;
    uint64_t fuel = 0;
    std::vector<WEntry> wlog;   /* this round's writes, one entry per cell, insertion order */
};

struct Access {          /* one in-bounds shared/global access, for X9 */
    uint32_t tlin;
    uint32_t gtid;
    int site;
    int arr;
    uint32_t addr;
    std::vector<uint32_t> iter;   /* counters of the site's enclosing loops */
};

struct Config {
    uint32_t bits = 32, input_mode = IN_RAND32, input_range = 0, checks = 0, bank_model = 0, wmax = 32;
    uint64_t fuel = 1u << 20;
    bool vcliteral = false;
    bool dataflow = false;
    uint32_t lock_rounds = 0;   /* lock-step comparison: snapshot rounds < lock_rounds (0: off) */
};

struct DFRow {   /* data-flow relation row (H5): who supplied the value of a read */
    uint32_t block, round, gtid, site, array, addr, src_kind, w_block, w_round, w_gtid;
};

/* Per-(launch,kernel) static information */
struct KInfo {
    const Kernel* K;
    Prog prog;
    std::vector<int> gid;    /* arr index -> global id across the pair (globals only) */
};

struct Runner {
    const Config& cfg;
    uint32_t mask;
    explicit Runner(const Config& c) : cfg(c) { mask = c.bits >= 32 ? 0xFFFFFFFFu : ((1u << c.bits) - 1u); }

    /* signed view of a w-bit value */
    int64_t sx(uint32_t v) const {
        if (cfg.bits >= 32) return (int64_t)(int32_t)v;
        uint32_t sign = 1u << (cfg.bits - 1);
        return (int64_t)(v ^ sign) - (int64_t)sign;
    }
    /* X2: w-bit two's-complement arithmetic; SMT-LIB division by zero */
    uint32_t binop(int op, int ty, uint32_t a, uint32_t b) const {
        const uint32_t w = cfg.bits;
        switch (op) {
        case B_ADD: return (a + b) & mask;
        case B_SUB: return (a - b) & mask;
        case B_MUL: return (uint32_t)((uint64_t)a * (uint64_t)b) & mask;
        case B_DIV:
            if (ty == TY_UNS) return b == 0 ? mask : (a / b) & mask;
            else {
                int64_t x = sx(a), y = sx(b);
                if (y == 0) return x < 0 ? 1u : mask;
                return (uint32_t)(uint64_t)(x / y) & mask;
            }
        case B_REM:
            if (ty == TY_UNS) return b == 0 ? a : (a % b) & mask;
            else {
                int64_t x = sx(a), y = sx(b);
                if (y == 0) return a;
                return (uint32_t)(uint64_t)(x % y) & mask;
            }
        case B_SHL: return b >= w ? 0u : (uint32_t)(((uint64_t)a << b) & mask);
        case B_SHR:
            if (ty == TY_UNS) return b >= w ? 0u : (a >> b);
            else {
                int64_t x = sx(a);
                if (b >= w) return x < 0 ? mask : 0u;
                return (uint32_t)(uint64_t)(x >> b) & mask;
            }
        case B_AND: return a & b;
        case B_OR: return a | b;
        case B_XOR: return a ^ b;
        case B_LT: return ty == TY_UNS ? (a < b) : (sx(a) < sx(b));
        case B_LE: return ty == TY_UNS ? (a <= b) : (sx(a) <= sx(b));
        case B_GT: return ty == TY_UNS ? (a > b) : (sx(a) > sx(b));
        case B_GE: return ty == TY_UNS ? (a >= b) : (sx(a) >= sx(b));
        case B_EQ: return a == b;
        case B_NE: return a != b;
        }
        throw Error(E_ARG, "internal: bad binop");
    }
};

/* Evaluate a uniform expression (array sizes / dims) with 32-bit arithmetic. */
static uint32_t eval_uniform(const Kernel& K, const Expr* e, const Launch& L) {
    Config c32;
    Runner R(c32);
    std::function<uint32_t(const Expr*)> ev = [&](const Expr* x) -> uint32_t {
        switch (x->k) {
        case EX_NUM: return x->num;
        case EX_VAR: {
            for (size_t i = 0; i < K.scalar_vars.size(); i++)
                if (K.scalar_vars[i] == x->var) return (uint32_t)L.scalar[i];
            throw Error(E_TYPE, at(x->line, x->col) + "size expression may only use scalars, bdim and gdim");
        }
        case EX_BUILTIN:
            if (x->bi >= BI_BDIM && x->bi < BI_BDIM + 3) return L.bdim[x->bi - BI_BDIM];
            if (x->bi >= BI_GDIM && x->bi < BI_GDIM + 3) return L.gdim[x->bi - BI_GDIM];
            throw Error(E_TYPE, at(x->line, x->col) + "size expression may only use scalars, bdim and gdim");
        case EX_NEG: return 0u - ev(x->a);
        case EX_BNOT: return ~ev(x->a);
        case EX_LNOT: return ev(x->a) == 0;
        case EX_CAST: return ev(x->a);
        case EX_LAND: return ev(x->a) ? (ev(x->b) != 0) : 0u;
        case EX_LOR: return ev(x->a) ? 1u : (ev(x->b) != 0);
        case EX_COND: return ev(x->a) ? ev(x->b) : ev(x->c);
        case EX_MIN: case EX_MAX: {
            uint32_t a = ev(x->a), b = ev(x->b);
            bool lt = R.binop(B_LT, x->opty, a, b);
            return (x->k == EX_MIN) == lt ? a : b;
        }
        case EX_BIN: return R.binop(x->op, x->opty, ev(x->a), ev(x->b));
        default: throw Error(E_TYPE, at(x->line, x->col) + "size expression may not read memory");
        }
    };
    return ev(e);
}

/* Lock-step comparison (X25): the contents of
 * one shared array of one block after one round, as (written << 32) | value. */
struct Snap {
    uint32_t block, round;
    std::string name;
    std::vector<uint64_t> cells;
};
struct DivRow {   /* first divergence of an instance: block, round, array, addr, values, written flags */
    uint32_t launch, seed_idx, block, round, array, addr, val_s, val_t, wr_s, wr_t;
};

struct Results {
    /* slots[(launch, seed_j, kernel)][kind] */
    std::map<std::tuple<uint32_t, uint32_t, uint32_t>, SlotSet> slots;
    uint64_t instances = 0;
    std::vector<uint64_t> site_stats;   /* [n_launch][stats_nk][max_sites][8] */
    uint32_t max_sites = 0, stats_nk = 2;
    std::vector<DFRow> df;
    std::vector<Snap> snaps[2];      /* per kernel, this instance */
    std::vector<DivRow> div;
};

/* Executes one kernel for one (launch, seed); returns final global memory. */
struct Exec {
    const Config& cfg;
    Runner R;
    const KInfo& KI;
    const Kernel& K;
    const Launch& L;
    uint64_t seed;
    uint32_t launch_idx, seed_idx, kernel_idx;
    Slot* slots;                    /* [N_KINDS] */
    Results& res;

    /* per-array runtime shape */
    std::vector<uint32_t> size;                  /* flat size per array */
    std::vector<std::vector<uint32_t>> dims;     /* dims per array */
    /* global memory (per instance) */
    std::vector<std::vector<uint32_t>> gval, glast, gfirst_blk, glast_blk;
    /* data-flow owner of each global cell: (block, round, gtid) of last commit */
    std::vector<std::vector<std::array<uint32_t, 3>>> gowner;
    /* shared memory (per block) */
    std::vector<std::vector<uint32_t>> sval;
    std::vector<std::vector<uint8_t>> swritten;
    std::vector<std::vector<std::array<uint32_t, 3>>> sowner;

    uint32_t T = 0, nblocks = 0;
    uint32_t cur_block = 0, cur_round = 0;
    uint32_t bid[3] = {0, 0, 0};
    std::vector<Thread> th;
    std::map<Cell, std::set<uint32_t>> readers;   /* this round: cell -> reader tlin */
    std::vector<Access> accesses;                 /* this round */
    /* VC-literal history (L521-L522, L598-L599, L709-L712): the state at the start of
       every round of this instance - each thread's registers and pc, the block's shared
       memory and the global memory - so that the guard p(s) and address e(s) of every
       write of thread s in that round can be re-evaluated on their own, independently of
       the write logs, commits and ownership tables of the execution being checked. */
    struct Hist {
        uint32_t block, round;
        std::vector<Thread> start;
        std::vector<std::vector<uint32_t>> sval, gval;
        std::vector<std::vector<uint8_t>> swritten;
        std::vector<std::vector<Cell>> wset;   /* per thread: cells it writes (lazily re-evaluated) */
        bool evaluated = false;
    };
    std::vector<Hist> hist;
    const Hist* shadow = nullptr;   /* non-null while re-evaluating a thread of that round */
    /* multi-kernel sequences (NEXT-4): the global buffers of the sequence so far, by pair-level
       id; a phase starts from them (buffers a phase is the first to use: PRF contents) and
       leaves its final contents there */
    std::map<uint32_t, std::vector<uint32_t>>* state = nullptr;

    Exec(const Config& c, const KInfo& ki, const Launch& l, uint64_t sd, uint32_t li, uint32_t si, uint32_t ki_,
         Slot* sl, Results& r)
        : cfg(c), R(c), KI(ki), K(*ki.K), L(l), seed(sd), launch_idx(li), seed_idx(si), kernel_idx(ki_),
          slots(sl), res(r) {}

    void event(int kind, uint32_t round, uint32_t arr, uint32_t addr, uint32_t ta, uint32_t tb, uint32_t site,
               uint32_t va, uint32_t vb) {
        if (shadow) return;   /* re-evaluation for the VC-literal check reports nothing */
        Ev e;
        e.f[0] = round; e.f[1] = arr; e.f[2] = addr; e.f[3] = ta; e.f[4] = tb; e.f[5] = site; e.f[6] = va; e.f[7] = vb;
        slots[kind].add(e);
    }
    uint32_t rec_arr_id(int a) const {
        const Arr& A = K.arrs[(size_t)a];
        if (A.space == SP_GLOBAL) return (uint32_t)KI.gid[(size_t)a];
        if (A.space == SP_SHARED) return 0x100u + (uint32_t)A.local_index;
        return 0x200u + (uint32_t)A.local_index;
    }
    /* X7/X8: initial contents of global array (pair id g), cell idx */
    uint32_t init_val(uint32_t g, uint32_t idx) const {
        uint32_t v;
        if (cfg.input_mode == IN_BITS01) v = idx < 64 ? (uint32_t)((seed >> idx) & 1u) : 0u;
        else if (cfg.input_mode == IN_RANGE) v = rand32(seed, g, idx) % (cfg.input_range ? cfg.input_range : 1u);
        else v = rand32(seed, g, idx);
        return v & R.mask;
    }
    /* X5/X6 poison values */
    uint32_t poison(int a, uint32_t addr) const {
        const Arr& A = K.arrs[(size_t)a];
        if (A.space == SP_GLOBAL) return rand32(seed, (uint64_t)KI.gid[(size_t)a], addr) & R.mask;
        uint64_t blin = cur_block;
        return rand32(seed, 0x8000u + (uint64_t)A.local_index, (blin << 20) + addr) & R.mask;
    }

    uint32_t builtin(const Thread& t, int bi) const {
        uint32_t v;
        if (bi < BI_BID) v = t.tid[bi - BI_TID];
        else if (bi < BI_BDIM) v = bid[bi - BI_BID];
        else if (bi < BI_GDIM) v = L.bdim[bi - BI_BDIM];
        else v = L.gdim[bi - BI_GDIM];
        return v & R.mask;
    }

    /* row-major flat index, 32-bit wrapping address arithmetic (X5) */
    uint32_t flat_index(int a, const std::vector<uint32_t>& iv) const {
        const std::vector<uint32_t>& d = dims[(size_t)a];
        uint32_t f = iv[0];
        for (size_t k = 1; k < iv.size(); k++) f = f * d[k] + iv[k];
        return f;
    }

    void record_access(const Thread& t, int site, int a, uint32_t addr) {
        if (shadow || !(cfg.checks & (CHK_BANK | CHK_COALESCE))) return;
        Access ac;
        ac.tlin = t.tlin; ac.gtid = t.gtid; ac.site = site; ac.arr = a; ac.addr = addr;
        for (int l : K.site_loops[(size_t)site]) ac.iter.push_back(t.loopctr[(size_t)l]);
        accesses.push_back(ac);
    }
    void mark_xb(int a, uint32_t addr) {
        if (shadow || K.arrs[(size_t)a].space != SP_GLOBAL) return;
        auto& f = gfirst_blk[(size_t)a];
        if (f[addr] == 0) f[addr] = cur_block + 1;
        glast_blk[(size_t)a][addr] = cur_block + 1;
    }

    /* Fig. 2 instantiation (L582-L599): for every thread s of round H, evaluate its
       segment alone from the round-start state - the values of its guards p(s) and write
       addresses e(s) - and keep the cells it writes.  Reads see the round-start memory
       plus s's own earlier writes (X3), exactly as in the paper's per-thread CA maps. */
    void literal_write_sets(Hist& H) {
        if (H.evaluated) return;
        const uint32_t blk = cur_block, b0 = bid[0], b1 = bid[1], b2 = bid[2];
        cur_block = H.block;
        bid[0] = H.block % L.gdim[0];
        bid[1] = (H.block / L.gdim[0]) % L.gdim[1];
        bid[2] = H.block / (L.gdim[0] * L.gdim[1]);
        shadow = &H;
        H.wset.assign(H.start.size(), {});
        for (size_t s = 0; s < H.start.size(); s++) {
            if (H.start[s].exited) continue;
            Thread t = H.start[s];
            t.wlog.clear();
            run_thread(t);
            for (const WEntry& w : t.wlog) H.wset[s].push_back(w.c);
        }
        shadow = nullptr;
        cur_block = blk;
        bid[0] = b0; bid[1] = b1; bid[2] = b2;
        H.evaluated = true;
    }

    /* VC-literal writer of cell c read in the current round: for every earlier round
       (latest first; shared cells: this block's rounds, global cells: every block run so
       far) enumerate all threads s and test p(s) ∧ c = e(s) on the re-evaluated maps
       (L521-L522, L709-L712); returns (found, block, round, min writer tlin).  More than one
       s is exactly a WW race (L517-L518). */
    bool vc_literal_writer(const Cell& c, bool global, uint32_t& wb, uint32_t& wr, uint32_t& wt) {
        for (size_t h = hist.size() - 1; h-- > 0;) {   /* (the last entry is the current round) */
            Hist& H = hist[h];
            if (!global && H.block != cur_block) continue;
            literal_write_sets(H);
            std::vector<uint32_t> S;
            for (uint32_t s = 0; s < (uint32_t)H.wset.size(); s++)
                for (const Cell& w : H.wset[s])
                    if (w == c) S.push_back(s);
            if (!S.empty()) {
                wb = H.block; wr = H.round; wt = *std::min_element(S.begin(), S.end());
                return true;
            }
        }
        return false;
    }

    /* a load while re-evaluating a thread for the VC-literal check: round-start memory */
    uint32_t shadow_load(Thread& t, int a, uint32_t f) {
        const Arr& A = K.arrs[(size_t)a];
        if (f >= size[(size_t)a]) return poison(a, f);
        Cell c{a, f};
        for (const WEntry& w : t.wlog)
            if (w.c == c) return w.val;
        if (A.space == SP_GLOBAL) return shadow->gval[(size_t)a][f];
        const size_t li = (size_t)A.local_index;
        return shadow->swritten[li][f] ? shadow->sval[li][f] : poison(a, f);
    }

    uint32_t load(Thread& t, const Expr* e) {
        std::vector<uint32_t> iv;
        for (Expr* x : e->idx) iv.push_back(eval(t, x));
        int a = e->arr;
        const Arr& A = K.arrs[(size_t)a];
        uint32_t f = flat_index(a, iv);
        if (A.space == SP_PRIVATE) {
            if (f >= size[(size_t)a]) {
                if (cfg.checks & CHK_OOB) event(K_OOB, cur_round, rec_arr_id(a), f, t.gtid, NONE32, (uint32_t)e->site, 0, 0);
                return 0;
            }
            return t.parr[(size_t)A.local_index][f];
        }
        if (shadow) return shadow_load(t, a, f);
        if (f >= size[(size_t)a]) {
            uint32_t pv = poison(a, f);
            if (cfg.checks & CHK_OOB) event(K_OOB, cur_round, rec_arr_id(a), f, t.gtid, NONE32, (uint32_t)e->site, pv, 0);
            return pv;
        }
        record_access(t, e->site, a, f);
        mark_xb(a, f);
        Cell c{a, f};
        readers[c].insert(t.tlin);
        for (const WEntry& w : t.wlog) {
            if (w.c == c) {
                if (cfg.dataflow)
                    res.df.push_back({cur_block, cur_round, t.gtid, (uint32_t)e->site, rec_arr_id(a), f, 2,
                                      cur_block, cur_round, t.gtid});
                return w.val;
            }
        }
        uint32_t v;
        std::array<uint32_t, 3> own{NONE32, NONE32, NONE32};
        if (A.space == SP_GLOBAL) {
            v = gval[(size_t)a][f];
            if (glast[(size_t)a][f]) own = gowner[(size_t)a][f];
        } else {
            if (!swritten[(size_t)A.local_index][f]) {
                v = poison(a, f);
                if (cfg.checks & CHK_OOB)
                    event(K_UNINIT, cur_round, rec_arr_id(a), f, t.gtid, NONE32, (uint32_t)e->site, v, 0);
            } else {
                v = sval[(size_t)A.local_index][f];
                own = sowner[(size_t)A.local_index][f];
            }
        }
        if (cfg.vcliteral) {
            uint32_t wb = NONE32, wr = NONE32, wt = NONE32;
            bool found = vc_literal_writer(c, A.space == SP_GLOBAL, wb, wr, wt);
            uint32_t wg = found ? wb * T + wt : NONE32;
            if (found != (own[0] != NONE32) || (found && (own[0] != wb || own[1] != wr || own[2] != wg)))
                throw Error(E_ARG, "VC-literal writer disagrees with ownership table at block " +
                                       std::to_string(cur_block) + " round " + std::to_string(cur_round));
        }
        if (cfg.dataflow)
            res.df.push_back({cur_block, cur_round, t.gtid, (uint32_t)e->site, rec_arr_id(a), f,
                              own[0] == NONE32 ? 0u : 1u, own[0], own[1], own[2]});
        return v;
    }

    void store(Thread& t, const Ins& in) {
        std::vector<uint32_t> iv;
        for (Expr* x : in.idx) iv.push_back(eval(t, x));
        uint32_t val = eval(t, in.e);
        int a = in.arr;
        const Arr& A = K.arrs[(size_t)a];
        uint32_t f = flat_index(a, iv);
        if (A.space == SP_PRIVATE) {
            if (f >= size[(size_t)a]) {
                if (cfg.checks & CHK_OOB) event(K_OOB, cur_round, rec_arr_id(a), f, t.gtid, NONE32, (uint32_t)in.site, val, 1);
                return;
            }
            t.parr[(size_t)A.local_index][f] = val;
            return;
        }
        if (f >= size[(size_t)a]) {   /* X5: OOB write is dropped */
            if (cfg.checks & CHK_OOB) event(K_OOB, cur_round, rec_arr_id(a), f, t.gtid, NONE32, (uint32_t)in.site, val, 1);
            return;
        }
        record_access(t, in.site, a, f);
        mark_xb(a, f);
        Cell c{a, f};
        for (WEntry& w : t.wlog) {
            if (w.c == c) { w.val = val; w.site = in.site; return; }
        }
        if (t.wlog.size() >= cfg.wmax) {   /* X19: write-log limit */
            event(K_LIMIT, cur_round, rec_arr_id(a), f, t.gtid, NONE32, (uint32_t)in.site, 1, 0);
            return;
        }
        t.wlog.push_back({c, val, in.site});
    }

    uint32_t eval(Thread& t, const Expr* e) {
        switch (e->k) {
        case EX_NUM: return e->num & R.mask;
        case EX_VAR: return t.vars[(size_t)e->var];
        case EX_BUILTIN: return builtin(t, e->bi);
        case EX_LOAD: return load(t, e);
        case EX_NEG: return (0u - eval(t, e->a)) & R.mask;
        case EX_BNOT: return (~eval(t, e->a)) & R.mask;
        case EX_LNOT: return eval(t, e->a) == 0 ? 1u : 0u;
        case EX_CAST: return eval(t, e->a);
        case EX_LAND: if (eval(t, e->a) == 0) return 0; return eval(t, e->b) != 0 ? 1u : 0u;
        case EX_LOR: if (eval(t, e->a) != 0) return 1; return eval(t, e->b) != 0 ? 1u : 0u;
        case EX_COND: return eval(t, e->a) != 0 ? eval(t, e->b) : eval(t, e->c);
        case EX_MIN: case EX_MAX: {
            uint32_t a = eval(t, e->a), b = eval(t, e->b);
            uint32_t lt = R.binop(B_LT, e->opty, a, b);
            if (e->k == EX_MIN) return lt ? a : b;
            return lt ? b : a;
        }
        case EX_BIN: {
            uint32_t a = eval(t, e->a);
            uint32_t b = eval(t, e->b);
            return R.binop(e->op, e->opty, a, b);
        }
        }
        throw Error(E_ARG, "internal: bad expression");
    }

    /* Run thread t from its pc until it reaches a barrier or exits. */
    void run_thread(Thread& t) {
        const std::vector<Ins>& P = KI.prog.ins;
        t.at_bar = false;
        t.fuel = 0;
        for (;;) {
            const Ins& in = P[(size_t)t.pc];
            switch (in.k) {
            case IN_ASSIGN: t.vars[(size_t)in.var] = eval(t, in.e); t.pc++; break;
            case IN_STORE: store(t, in); t.pc++; break;
            case IN_PDECL: {
                const Arr& A = K.arrs[(size_t)in.arr];
                std::fill(t.parr[(size_t)A.local_index].begin(), t.parr[(size_t)A.local_index].end(), 0u);
                t.pc++;
                break;
            }
            case IN_JZ: t.pc = eval(t, in.e) == 0 ? in.target : t.pc + 1; break;
            case IN_JMP: t.pc = in.target; break;
            case IN_SYNC: t.at_bar = true; t.bar_site = in.site; t.pc++; return;
            case IN_RET: case IN_END: t.exited = true; return;
            case IN_LENTER: t.loopctr[(size_t)in.loop_id] = 0; t.pc++; break;
            case IN_LNEXT:
                t.loopctr[(size_t)in.loop_id]++;
                if (++t.fuel > cfg.fuel) {   /* X19: loop fuel per thread per round */
                    event(K_LIMIT, cur_round, NONE32, 0, t.gtid, NONE32, NONE32, 2, 0);
                    t.exited = true;
                    return;
                }
                t.pc++;
                break;
            default: throw Error(E_ARG, "internal: bad instruction");
            }
        }
    }

    /* X9: bank / coalescing statistics of this round's accesses */
    void bank_stats() {
        if (accesses.empty()) return;
        /* group by (warp, site, iteration vector) */
        std::map<std::tuple<uint32_t, int, std::vector<uint32_t>>, std::vector<const Access*>> groups;
        for (const Access& ac : accesses) {
            const Arr& A = K.arrs[(size_t)ac.arr];
            uint32_t wsz = (A.space == SP_SHARED && cfg.bank_model == 1) ? 16u : 32u;
            groups[std::make_tuple(ac.tlin / wsz, ac.site, ac.iter)].push_back(&ac);
        }
        for (auto& g : groups) {
            const std::vector<const Access*>& v = g.second;
            int site = std::get<1>(g.first);
            int a = v[0]->arr;
            const Arr& A = K.arrs[(size_t)a];
            uint64_t* st = nullptr;
            if (site < (int)res.max_sites)
                st = &res.site_stats[(((size_t)launch_idx * res.stats_nk + kernel_idx) * res.max_sites + (size_t)site) * 8];
            if (A.space == SP_SHARED) {
                if (!(cfg.checks & CHK_BANK)) continue;
                uint32_t nb = cfg.bank_model == 1 ? 16u : 32u;
                std::map<uint32_t, std::set<uint32_t>> bankwords;
                for (const Access* x : v) bankwords[x->addr % nb].insert(x->addr);
                uint32_t deg = 0, bstar = 0;
                for (auto& bw : bankwords)
                    if ((uint32_t)bw.second.size() > deg) { deg = (uint32_t)bw.second.size(); bstar = bw.first; }
                if (st) {   /* [space, n_acc, n_bad, max, sum, sum_ideal, sum_lanes, 0] */
                    st[0] = 1; st[1] += 1; st[2] += deg > 1; st[3] = std::max<uint64_t>(st[3], deg); st[4] += deg;
                    st[5] += 1; st[6] += v.size();
                }
                if (deg > 1) {
                    uint32_t astar = *bankwords[bstar].begin();
                    uint32_t ta = NONE32, tb = NONE32;
                    for (const Access* x : v) {
                        if (x->addr == astar) ta = std::min(ta, x->gtid);
                        else if (x->addr % nb == bstar) tb = std::min(tb, x->gtid);
                    }
                    event(K_BANK, cur_round, rec_arr_id(a), astar, ta, tb, (uint32_t)site, deg, 0);
                }
            } else {
                if (!(cfg.checks & CHK_COALESCE)) continue;
                std::set<uint32_t> words, sectors;
                uint32_t amin = NONE32, ta = NONE32, tb = 0;
                for (const Access* x : v) {
                    words.insert(x->addr);
                    sectors.insert(x->addr >> 3);   /* 32-byte sectors of 4-byte words, 256B-aligned base */
                    amin = std::min(amin, x->addr);
                    ta = std::min(ta, x->gtid);
                    tb = std::max(tb, x->gtid);
                }
                uint32_t S = (uint32_t)sectors.size();
                uint32_t ideal = ((uint32_t)words.size() + 7u) / 8u;
                if (st) {
                    st[0] = 2; st[1] += 1; st[2] += S > ideal; st[3] = std::max<uint64_t>(st[3], S); st[4] += S;
                    st[5] += ideal; st[6] += v.size();
                }
                if (S > ideal) event(K_UNCOALESCED, cur_round, rec_arr_id(a), amin, ta, tb, (uint32_t)site, S, ideal);
            }
        }
        accesses.clear();
    }

    /* X3/X4: commit this round's writes; report WW and RW races */
    void commit_round() {
        std::map<Cell, std::vector<uint32_t>> writers;   /* cell -> writer tlins (ascending: threads visited in order) */
        for (uint32_t i = 0; i < T; i++)
            for (const WEntry& w : th[i].wlog) writers[w.c].push_back(i);
        for (auto& cw : writers) {
            const Cell& c = cw.first;
            const std::vector<uint32_t>& W = cw.second;
            uint32_t w0 = W.front(), w1 = W.back();
            auto val_of = [&](uint32_t tl, int* site) -> uint32_t {
                for (const WEntry& w : th[tl].wlog) if (w.c == c) { if (site) *site = w.site; return w.val; }
                throw Error(E_ARG, "internal: missing log entry");
            };
            int site0 = -1;
            uint32_t v0 = val_of(w0, &site0);
            const Arr& A = K.arrs[(size_t)c.arr];
            uint32_t gw0 = cur_block * T + w0;
            if (A.space == SP_GLOBAL) {
                gval[(size_t)c.arr][c.addr] = v0;
                glast[(size_t)c.arr][c.addr] = gw0 + 1;
                gowner[(size_t)c.arr][c.addr] = {cur_block, cur_round, gw0};
            } else {
                sval[(size_t)A.local_index][c.addr] = v0;
                swritten[(size_t)A.local_index][c.addr] = 1;
                sowner[(size_t)A.local_index][c.addr] = {cur_block, cur_round, gw0};
            }
            if (!(cfg.checks & CHK_RACE)) continue;
            if (w1 != w0)   /* X16: (min writer, max writer), the committed write's site and value */
                event(K_RACE_WW, cur_round, rec_arr_id(c.arr), c.addr, gw0, cur_block * T + w1, (uint32_t)site0, v0,
                      0);
            auto rit = readers.find(c);
            if (rit != readers.end() && !rit->second.empty()) {
                uint32_t rmin = *rit->second.begin(), rmax = *rit->second.rbegin();
                if (!(rmin == rmax && w0 == w1 && rmin == w0)) {
                    uint32_t ta, tb;
                    if (rmin != w0) { ta = w0; tb = rmin; }
                    else if (rmax != w0) { ta = w0; tb = rmax; }
                    else { ta = w1; tb = rmin; }
                    int sa = -1;
                    uint32_t va = val_of(ta, &sa);
                    event(K_RACE_RW, cur_round, rec_arr_id(c.arr), c.addr, cur_block * T + ta, cur_block * T + tb,
                          (uint32_t)sa, va, 0);
                }
            }
        }
    }

    void run() {
        T = L.bdim[0] * L.bdim[1] * L.bdim[2];
        nblocks = L.gdim[0] * L.gdim[1] * L.gdim[2];
        size.assign(K.arrs.size(), 0);
        dims.assign(K.arrs.size(), {});
        for (size_t a = 0; a < K.arrs.size(); a++) {
            const Arr& A = K.arrs[a];
            uint64_t s = 1;
            for (const Expr* d : A.dims) {
                uint32_t dv = eval_uniform(K, d, L);
                dims[a].push_back(dv);
                s *= dv;
                if (s > (1u << 24)) throw Error(E_LIMIT, "array '" + A.name + "' larger than 2^24 words");
            }
            size[a] = (uint32_t)s;
        }
        gval.assign(K.arrs.size(), {}); glast.assign(K.arrs.size(), {});
        gfirst_blk.assign(K.arrs.size(), {}); glast_blk.assign(K.arrs.size(), {});
        gowner.assign(K.arrs.size(), {});
        for (size_t a = 0; a < K.arrs.size(); a++) {
            if (K.arrs[a].space != SP_GLOBAL) continue;
            gval[a].resize(size[a]);
            const uint32_t g = (uint32_t)KI.gid[a];
            if (state) {   /* sequence: the buffer as the previous phases left it */
                std::vector<uint32_t>& b = (*state)[g];
                for (uint32_t i = (uint32_t)b.size(); i < size[a]; i++) b.push_back(init_val(g, i));
                for (uint32_t i = 0; i < size[a]; i++) gval[a][i] = b[i];
            } else {
                for (uint32_t i = 0; i < size[a]; i++) gval[a][i] = init_val(g, i);
            }
            glast[a].assign(size[a], 0);
            gfirst_blk[a].assign(size[a], 0);
            glast_blk[a].assign(size[a], 0);
            gowner[a].assign(size[a], {NONE32, NONE32, NONE32});
        }
        int nsh = 0, npr = 0;
        for (auto& A : K.arrs) { if (A.space == SP_SHARED) nsh++; if (A.space == SP_PRIVATE) npr++; }
        hist.clear();
        for (uint32_t b = 0; b < nblocks; b++) {
            cur_block = b;
            bid[0] = b % L.gdim[0];
            bid[1] = (b / L.gdim[0]) % L.gdim[1];
            bid[2] = b / (L.gdim[0] * L.gdim[1]);
            sval.assign((size_t)nsh, {}); swritten.assign((size_t)nsh, {}); sowner.assign((size_t)nsh, {});
            for (size_t a = 0; a < K.arrs.size(); a++) {
                const Arr& A = K.arrs[a];
                if (A.space != SP_SHARED) continue;
                sval[(size_t)A.local_index].assign(size[a], 0);
                swritten[(size_t)A.local_index].assign(size[a], 0);
                sowner[(size_t)A.local_index].assign(size[a], {NONE32, NONE32, NONE32});
            }
            th.assign(T, Thread());
            for (uint32_t i = 0; i < T; i++) {
                Thread& t = th[i];
                t.tid[0] = i % L.bdim[0];
                t.tid[1] = (i / L.bdim[0]) % L.bdim[1];
                t.tid[2] = i / (L.bdim[0] * L.bdim[1]);
                t.tlin = i;
                t.gtid = b * T + i;
                t.vars.assign(K.vars.size(), 0);
                for (size_t s = 0; s < K.scalar_vars.size(); s++)
                    t.vars[(size_t)K.scalar_vars[s]] = (uint32_t)L.scalar[s] & R.mask;
                t.parr.assign((size_t)npr, {});
                for (size_t a = 0; a < K.arrs.size(); a++)
                    if (K.arrs[a].space == SP_PRIVATE) t.parr[(size_t)K.arrs[a].local_index].assign(size[a], 0);
                t.loopctr.assign((size_t)K.n_loops, 0);
            }
            cur_round = 0;
            for (;;) {
                readers.clear();
                for (uint32_t i = 0; i < T; i++) th[i].wlog.clear();
                if (cfg.vcliteral) {   /* round-start state for the literal re-evaluation */
                    Hist H;
                    H.block = b; H.round = cur_round; H.start = th; H.sval = sval; H.swritten = swritten;
                    H.gval = gval;
                    hist.push_back(std::move(H));
                }
                /* natural order, L384-L389 */
                for (uint32_t i = 0; i < T; i++)
                    if (!th[i].exited) run_thread(th[i]);
                /* X18: barrier divergence */
                std::map<int, uint32_t> sites;   /* barrier site -> lowest thread waiting there */
                for (uint32_t i = 0; i < T; i++)
                    if (!th[i].exited && th[i].at_bar && !sites.count(th[i].bar_site)) sites[th[i].bar_site] = i;
                if (sites.size() > 1) {
                    auto it = sites.begin();
                    int s0 = it->first; uint32_t t0 = it->second;
                    ++it;
                    event(K_BARRIER_DIV, cur_round, NONE32, 0, b * T + t0, b * T + it->second, (uint32_t)s0,
                          (uint32_t)it->first, 0);
                }
                commit_round();
                bank_stats();
                if (cur_round < cfg.lock_rounds) {   /* X25: shared state after this round */
                    for (size_t a = 0; a < K.arrs.size(); a++) {
                        const Arr& A = K.arrs[a];
                        if (A.space != SP_SHARED) continue;
                        Snap sn;
                        sn.block = b; sn.round = cur_round; sn.name = A.name;
                        const size_t li = (size_t)A.local_index;
                        for (uint32_t i = 0; i < size[a]; i++)
                            sn.cells.push_back(swritten[li][i] ? ((1ull << 32) | sval[li][i]) : 0ull);
                        res.snaps[kernel_idx].push_back(std::move(sn));
                    }
                }
                bool any = false;
                for (uint32_t i = 0; i < T; i++) any |= !th[i].exited;
                cur_round++;
                if (!any) break;
                if (cur_round >= ROUND_LIMIT) {   /* X19: the round field saturates (X16 keys keep 16 bits) */
                    for (uint32_t i = 0; i < T; i++)
                        if (!th[i].exited) {
                            event(K_LIMIT, ROUND_LIMIT, NONE32, 0, b * T + i, NONE32, NONE32, 3, 0);
                            th[i].exited = true;
                        }
                    break;
                }
            }
            res.instances += (uint64_t)T * cur_round;   /* X19: threads x rounds per block */
        }
        if (state)   /* sequence: the phase's final contents stay in the buffers */
            for (size_t a = 0; a < K.arrs.size(); a++)
                if (K.arrs[a].space == SP_GLOBAL) {
                    std::vector<uint32_t>& b = (*state)[(uint32_t)KI.gid[a]];
                    for (uint32_t i = 0; i < size[a]; i++) b[i] = gval[a][i];
                }
        /* X4: cross-block races on global cells */
        if (cfg.checks & CHK_RACE) {
            for (size_t a = 0; a < K.arrs.size(); a++) {
                if (K.arrs[a].space != SP_GLOBAL) continue;
                for (uint32_t i = 0; i < size[a]; i++) {
                    if (glast[a][i] && gfirst_blk[a][i] != glast_blk[a][i])
                        event(K_RACE_XB, ROUND_END, rec_arr_id((int)a), i, gfirst_blk[a][i] - 1, glast_blk[a][i] - 1,
                              NONE32, gval[a][i], 0);
                }
            }
        }
    }
};

static std::unique_ptr<Kernel> parse_kernel(const std::string& text) {
    std::unique_ptr<Kernel> K(new Kernel());
    Parser P(text, K.get());
    P.kernel();
    return K;
}

/* ------------------------------------------------------------------ driver */
struct Space {
    const Launch* launch_src;
    const Launch* launch_tgt;
    uint32_t n_launch;
    uint64_t seed_base;
    uint32_t n_seeds;
    uint32_t rank, world;
    Config cfg;
    uint32_t mode;
};

static void check_launch(const Kernel& K, const Launch& L) {
    for (int d = 0; d < 3; d++)
        if (L.gdim[d] == 0 || L.bdim[d] == 0) throw Error(E_ARG, "zero launch dimension");
    uint64_t T = (uint64_t)L.bdim[0] * L.bdim[1] * L.bdim[2];
    if (T > 4096) throw Error(E_LIMIT, "more than 4096 threads per block");
    uint64_t G = (uint64_t)L.gdim[0] * L.gdim[1] * L.gdim[2];
    if (G > (1u << 20)) throw Error(E_LIMIT, "more than 2^20 blocks");
    if (L.n_scalar != K.scalar_vars.size()) throw Error(E_ARG, "scalar count does not match kernel '" + K.name + "'");
}

/* X25: the first (block, round, array, addr) - array in the source kernel's shared
 * declaration order - at which the two kernels' shared contents differ, over the
 * (block, round, array) snapshots both kernels took with the same array name and size. */
static void lockstep_compare(const Kernel& ks, uint32_t li, uint32_t sj, Results& res) {
    std::map<std::tuple<uint32_t, uint32_t, std::string>, const Snap*> tgt;
    for (const Snap& s : res.snaps[1]) tgt[std::make_tuple(s.block, s.round, s.name)] = &s;
    std::map<std::string, uint32_t> slot;   /* source shared array name -> record array id */
    for (const Arr& A : ks.arrs)
        if (A.space == SP_SHARED) slot[A.name] = 0x100u + (uint32_t)A.local_index;
    bool found = false;
    DivRow best{};
    for (const Snap& s : res.snaps[0]) {
        auto it = tgt.find(std::make_tuple(s.block, s.round, s.name));
        if (it == tgt.end() || it->second->cells.size() != s.cells.size()) continue;
        for (uint32_t i = 0; i < s.cells.size(); i++) {
            uint64_t a = s.cells[i], b = it->second->cells[i];
            if (a == b) continue;
            DivRow r{li, sj, s.block, s.round, slot[s.name], i, (uint32_t)a, (uint32_t)b,
                     (uint32_t)(a >> 32), (uint32_t)(b >> 32)};
            auto k = [](const DivRow& x) { return std::make_tuple(x.block, x.round, x.array, x.addr); };
            if (!found || k(r) < k(best)) best = r;
            found = true;
            break;   /* later cells of this snapshot are larger in the order */
        }
    }
    if (found) res.div.push_back(best);
}

/* The kernels of one check over the space: each is run once per (launch, seed); with two
 * or more, the comparative assertion (L441-L444, L652-L657) on every pair i < j, over every
 * global array that is out/inout in either kernel (matched by name).  A mismatch of the pair
 * is an event in slot (instance, kernel i, MISMATCH); its site field names j in N-kernel
 * checks (nmode) and is NONE for the two-kernel check. */
static void run_seq(const std::vector<const Kernel*>& kk, const std::vector<KInfo>& ki,
                    const std::vector<const Launch*>& lists, const Space& S, Results& res, uint32_t n_src);

static void run_space(const std::vector<const Kernel*>& kk, const std::vector<const Launch*>& lists, const Space& S,
                      Results& res, bool nmode, uint32_t seq_src = 0) {
    const int nk = (int)kk.size();
    std::vector<KInfo> ki((size_t)nk);
    /* X8: global ids = index in the sorted union of the kernels' global-array names */
    std::vector<std::string> names;
    for (int k = 0; k < nk; k++)
        for (auto& A : kk[k]->arrs) if (A.space == SP_GLOBAL) names.push_back(A.name);
    std::sort(names.begin(), names.end());
    names.erase(std::unique(names.begin(), names.end()), names.end());
    for (int k = 0; k < nk; k++) {
        ki[k].K = kk[k];
        Lowerer lw(ki[k].prog);
        lw.lower(kk[k]->body);
        Ins end; end.k = IN_END;
        ki[k].prog.ins.push_back(end);
        ki[k].gid.assign(kk[k]->arrs.size(), -1);
        for (size_t a = 0; a < kk[k]->arrs.size(); a++)
            if (kk[k]->arrs[a].space == SP_GLOBAL)
                ki[k].gid[a] = (int)(std::lower_bound(names.begin(), names.end(), kk[k]->arrs[a].name) - names.begin());
    }
    if (seq_src) {
        run_seq(kk, ki, lists, S, res, seq_src);
        return;
    }
    for (uint32_t li = 0; li < S.n_launch; li++) {
        std::vector<const Launch*> LL((size_t)nk);
        for (int k = 0; k < nk; k++) {
            LL[k] = &lists[k][li];
            check_launch(*kk[k], *LL[k]);
        }
        for (uint32_t sj = S.rank; sj < S.n_seeds; sj += S.world) {
            uint64_t seed = S.seed_base + sj;
            std::vector<std::vector<std::vector<uint32_t>>> fin((size_t)nk), flast((size_t)nk);
            std::vector<std::vector<uint32_t>> fsz((size_t)nk);
            res.snaps[0].clear();
            res.snaps[1].clear();
            for (int k = 0; k < nk; k++) {
                Slot* sl = res.slots[std::make_tuple(li, sj, (uint32_t)k)].s;
                Exec ex(S.cfg, ki[k], *LL[k], seed, li, sj, (uint32_t)k, sl, res);
                ex.run();
                fin[k] = ex.gval;
                flast[k] = ex.glast;
                fsz[k] = ex.size;
            }
            if (nk == 2 && S.cfg.lock_rounds) lockstep_compare(*kk[0], li, sj, res);
            if (nk < 2 || !(S.cfg.checks & CHK_EQUIV)) continue;
            for (int i = 0; i < nk; i++) {
                Slot* sl = res.slots[std::make_tuple(li, sj, (uint32_t)i)].s;
                for (int j = i + 1; j < nk; j++) {
                    for (size_t as = 0; as < kk[i]->arrs.size(); as++) {
                        const Arr& A = kk[i]->arrs[as];
                        if (A.space != SP_GLOBAL) continue;
                        for (size_t at_ = 0; at_ < kk[j]->arrs.size(); at_++) {
                            const Arr& B = kk[j]->arrs[at_];
                            if (B.space != SP_GLOBAL || B.name != A.name) continue;
                            if (A.mode == M_IN && B.mode == M_IN) continue;
                            uint32_t n = std::min(fsz[i][as], fsz[j][at_]);
                            for (uint32_t c = 0; c < n; c++) {
                                uint32_t va = fin[i][as][c], vb = fin[j][at_][c];
                                if (va != vb) {
                                    Ev e;
                                    uint32_t f[8] = {ROUND_END, (uint32_t)ki[i].gid[as], c, flast[i][as][c] - 1,
                                                     flast[j][at_][c] - 1, nmode ? (uint32_t)j : NONE32, va, vb};
                                    memcpy(e.f, f, sizeof f);
                                    sl[K_MISMATCH].add(e);
                                }
                            }
                        }
                    }
                }
            }
        }
    }
}

/* Multi-kernel sequences (GKLEE's multi-kernel programs L62-L63):
 * kernels 0..n_src-1 are the source sequence, n_src.. the target sequence.  Per (launch,
 * seed) each side runs its phases in order on ONE set of global buffers, matched by name
 * (a kernel boundary is a grid-wide barrier: every block of phase i finishes before phase
 * i+1 starts); a buffer's initial contents are the PRF's (X7/X8), its size the largest any
 * phase declares, each phase checking bounds against its own declaration (X5).  Races, OOB,
 * LIMIT, BARRIER_DIV per phase (record kernel = phase index).  The comparative assertion
 * compares the two sides' final buffers on every name both sides use and some phase writes
 * (out / inout): MISMATCH in kernel 0's slot, tid fields = the last writer in the side's
 * LAST phase (NONE if that phase did not write the cell). */
static void run_seq(const std::vector<const Kernel*>& kk, const std::vector<KInfo>& ki,
                    const std::vector<const Launch*>& lists, const Space& S, Results& res, uint32_t n_src) {
    const uint32_t nk = (uint32_t)kk.size();
    for (uint32_t li = 0; li < S.n_launch; li++) {
        for (uint32_t k = 0; k < nk; k++) check_launch(*kk[k], lists[k][li]);
        for (uint32_t sj = S.rank; sj < S.n_seeds; sj += S.world) {
            const uint64_t seed = S.seed_base + sj;
            std::map<uint32_t, std::vector<uint32_t>> state[2];
            std::map<uint32_t, std::vector<uint32_t>> last[2];   /* gid -> last writer + 1 in the side's last phase */
            std::map<uint32_t, bool> written[2];
            for (uint32_t k = 0; k < nk; k++) {
                const uint32_t side = k < n_src ? 0u : 1u;
                Slot* sl = res.slots[std::make_tuple(li, sj, k)].s;
                Exec ex(S.cfg, ki[k], lists[k][li], seed, li, sj, k, sl, res);
                ex.state = &state[side];
                ex.run();
                const bool last_phase = k == n_src - 1 || k == nk - 1;
                for (size_t a = 0; a < kk[k]->arrs.size(); a++) {
                    const Arr& A = kk[k]->arrs[a];
                    if (A.space != SP_GLOBAL) continue;
                    const uint32_t g = (uint32_t)ki[k].gid[a];
                    if (A.mode != M_IN) written[side][g] = true;
                    if (last_phase) last[side][g] = ex.glast[a];
                }
            }
            if (!(S.cfg.checks & CHK_EQUIV)) continue;
            Slot* sl = res.slots[std::make_tuple(li, sj, 0u)].s;
            for (auto& kv : state[0]) {
                const uint32_t g = kv.first;
                if (!state[1].count(g) || !(written[0][g] || written[1][g])) continue;
                const std::vector<uint32_t>& a = kv.second;
                const std::vector<uint32_t>& b = state[1][g];
                const uint32_t n = (uint32_t)std::min(a.size(), b.size());
                for (uint32_t c = 0; c < n; c++) {
                    if (a[c] == b[c]) continue;
                    auto lw = [&](int side) -> uint32_t {
                        auto it = last[side].find(g);
                        return it != last[side].end() && c < it->second.size() ? it->second[c] - 1 : NONE32;
                    };
                    Ev e;
                    uint32_t f[8] = {ROUND_END, g, c, lw(0), lw(1), NONE32, a[c], b[c]};
                    memcpy(e.f, f, sizeof f);
                    sl[K_MISMATCH].add(e);
                }
            }
        }
    }
}

}  // namespace orc

/* ------------------------------------------------------------------ C API  */
extern "C" {

typedef struct {
    uint32_t gdim[3], bdim[3];
    int32_t scalar[8];
    uint32_t n_scalar;
} or_launch;

typedef struct {
    uint64_t key, count;
    uint32_t kind, launch, seed_idx, kernel, round, site, array, addr, tid_a, tid_b, val_a, val_b;
} or_rec;

typedef struct {
    const or_launch* launch_src;
    const or_launch* launch_tgt;   /* NULL: same as launch_src */
    uint32_t n_launch;
    uint64_t seed_base;
    uint32_t n_seeds;
    uint32_t rank, world;
    uint32_t input_mode, input_range, bits, checks, bank_model, wmax;
    uint32_t mode;                 /* 0 equiv, 1 races, 2 banks */
    uint32_t vcliteral;
    uint32_t max_sites;            /* rows of site_stats per (launch, kernel) */
} or_space;

static thread_local std::string or_err;

const char* or_last_error(void) { return or_err.c_str(); }

/* The kernels texts[0..nk) over the space, the launches of kernel k in lists[k] (shared by
 * or_check and or_check_n). */
static int check_common(const char* const* texts, uint32_t nk, const or_launch* const* lists, bool nmode,
                        const or_space* sp, or_rec* recs, uint64_t cap, uint64_t* n_recs, int64_t* counts,
                        int64_t* first_key, uint64_t* site_stats, uint32_t seq_src = 0) {
    using namespace orc;
    try {
        if (!texts || !sp || !n_recs || !counts || !first_key || nk < 1 || nk > 8) throw Error(E_ARG, "null argument");
        for (uint32_t k = 0; k < nk; k++)
            if (!texts[k]) throw Error(E_ARG, "null kernel");
        if (sp->world == 0 || sp->rank >= sp->world) throw Error(E_ARG, "bad rank/world");
        if (sp->bits < 1 || sp->bits > 32) throw Error(E_ARG, "bits must be 1..32");
        if (sp->n_launch >= (1u << 18)) throw Error(E_LIMIT, "too many launches");
        if (sp->n_seeds >= (1u << 21)) throw Error(E_LIMIT, "too many seeds");
        std::vector<std::unique_ptr<Kernel>> ks;
        std::vector<const Kernel*> kk;
        std::vector<const Launch*> ll;
        static_assert(sizeof(or_launch) == sizeof(Launch), "launch layout");
        for (uint32_t k = 0; k < nk; k++) {
            ks.push_back(parse_kernel(texts[k]));
            kk.push_back(ks.back().get());
            ll.push_back(reinterpret_cast<const Launch*>(lists[k]));
        }
        Space S;
        S.launch_src = ll[0];
        S.launch_tgt = nk > 1 ? ll[1] : nullptr;
        S.n_launch = sp->n_launch;
        S.seed_base = sp->seed_base;
        S.n_seeds = sp->n_seeds;
        S.rank = sp->rank;
        S.world = sp->world;
        S.cfg.bits = sp->bits;
        S.cfg.input_mode = sp->input_mode;
        S.cfg.input_range = sp->input_range;
        S.cfg.checks = sp->checks;
        S.cfg.bank_model = sp->bank_model;
        S.cfg.wmax = sp->wmax ? sp->wmax : 32;
        S.cfg.vcliteral = sp->vcliteral != 0;
        S.mode = sp->mode;
        Results res;
        res.max_sites = site_stats ? sp->max_sites : 0;
        res.stats_nk = std::max<uint32_t>(2, nk);
        res.site_stats.assign((size_t)sp->n_launch * res.stats_nk * res.max_sites * 8, 0);
        run_space(kk, ll, S, res, nmode, seq_src);
        for (int i = 0; i < 16; i++) counts[i] = 0;
        for (int i = 0; i < 11; i++) first_key[i] = INT64_MAX;
        counts[0] = (int64_t)res.instances;
        uint64_t n = 0;
        std::set<std::pair<uint32_t, uint32_t>> failing_inst;
        for (auto& kv : res.slots) {   /* std::map iterates in (launch, seed, kernel) order */
            uint32_t li = std::get<0>(kv.first), sj = std::get<1>(kv.first), k = std::get<2>(kv.first);
            for (uint32_t kind = 0; kind < N_KINDS; kind++) {
                const Slot& s = kv.second.s[kind];
                if (!s.has) continue;
                uint64_t key = make_key(li, sj, k, kind, s.best.f[0]);
                counts[1 + kind] += (int64_t)s.count;
                bool failing = kind <= K_MISMATCH || kind == K_LIMIT ||
                               (sp->mode == MODE_BANKS && (kind == K_BANK || kind == K_UNCOALESCED));
                if ((int64_t)key < first_key[1 + kind]) first_key[1 + kind] = (int64_t)key;
                if (failing) {
                    if ((int64_t)key < first_key[0]) first_key[0] = (int64_t)key;
                    failing_inst.insert({li, sj});
                }
                if (n < cap && recs) {
                    or_rec& r = recs[n];
                    r.key = key; r.count = s.count; r.kind = kind; r.launch = li; r.seed_idx = sj; r.kernel = k;
                    r.round = s.best.f[0]; r.array = s.best.f[1]; r.addr = s.best.f[2]; r.tid_a = s.best.f[3];
                    r.tid_b = s.best.f[4]; r.site = s.best.f[5]; r.val_a = s.best.f[6]; r.val_b = s.best.f[7];
                }
                n++;
            }
        }
        counts[11] = (int64_t)n;
        counts[12] = (int64_t)failing_inst.size();
        *n_recs = n;
        if (site_stats) memcpy(site_stats, res.site_stats.data(), res.site_stats.size() * sizeof(uint64_t));
        return 0;
    } catch (const orc::Error& e) {
        or_err = e.what();
        return e.code;
    } catch (const std::exception& e) {
        or_err = e.what();
        return -1;
    }
}

/* Check a pair (tgt != NULL) or a single kernel over the space.
 * recs: caller buffer of cap records (canonical order); counts[16]; first_key[11];
 * site_stats: NULL or uint64[n_launch][2][max_sites][8] =
 *   [space (1 shared, 2 global), warp-accesses, conflicted|uncoalesced, max degree|sectors,
 *    sum degree|sectors, sum ideal, sum active lanes, 0]. */
int or_check(const char* src, const char* tgt, const or_space* sp, or_rec* recs, uint64_t cap, uint64_t* n_recs,
             int64_t* counts, int64_t* first_key, uint64_t* site_stats) {
    if (!sp) return -1;
    const char* texts[2] = {src, tgt};
    const or_launch* lists[2] = {sp->launch_src, sp->launch_tgt ? sp->launch_tgt : sp->launch_src};
    return check_common(texts, tgt ? 2u : 1u, lists, false, sp, recs, cap, n_recs, counts, first_key, site_stats);
}

/* N-kernel check (nk in 1..8): every kernel once per (launch, seed), launches[k] its launch
 * list (n_launch each, the same points n); the comparative assertion on every pair i < j,
 * MISMATCH records in the slot of kernel i with site = j.  site_stats: [n_launch][max(2,nk)]
 * [max_sites][8]. */
int or_check_n(const char* const* texts, uint32_t nk, const or_launch* const* launches, const or_space* sp,
               or_rec* recs, uint64_t cap, uint64_t* n_recs, int64_t* counts, int64_t* first_key,
               uint64_t* site_stats) {
    return check_common(texts, nk, launches, true, sp, recs, cap, n_recs, counts, first_key, site_stats);
}

/* Multi-kernel sequences: texts[0..n_src) the source sequence, texts[n_src..nk) the target
 * sequence (run_seq).  n_src >= 1, nk - n_src >= 1, nk <= 8. */
int or_check_seq(const char* const* texts, uint32_t nk, uint32_t n_src, const or_launch* const* launches,
                 const or_space* sp, or_rec* recs, uint64_t cap, uint64_t* n_recs, int64_t* counts,
                 int64_t* first_key) {
    if (n_src < 1 || n_src >= nk) {
        or_err = "a sequence check needs at least one kernel on each side";
        return -1;
    }
    return check_common(texts, nk, launches, false, sp, recs, cap, n_recs, counts, first_key, nullptr, n_src);
}

/* Run one kernel for one launch/seed and return its initial and final global
 * arrays, concatenated in global-id order (sorted names of this kernel).
 * sizes[i] receives the size of array i; returns the number of arrays. */
int or_exec(const char* text, const or_launch* launch, uint64_t seed, uint32_t input_mode, uint32_t input_range,
            uint32_t bits, uint32_t checks, uint32_t wmax, uint32_t* init_out, uint32_t* final_out, uint64_t cap, uint32_t* sizes,
            uint32_t max_arrays, uint32_t* n_arrays, int64_t* counts) {
    using namespace orc;
    try {
        std::unique_ptr<Kernel> K = parse_kernel(text);
        check_launch(*K, *reinterpret_cast<const Launch*>(launch));
        KInfo ki;
        ki.K = K.get();
        Lowerer lw(ki.prog);
        lw.lower(K->body);
        Ins end; end.k = IN_END;
        ki.prog.ins.push_back(end);
        std::vector<std::string> names;
        for (auto& A : K->arrs) if (A.space == SP_GLOBAL) names.push_back(A.name);
        std::sort(names.begin(), names.end());
        ki.gid.assign(K->arrs.size(), -1);
        for (size_t a = 0; a < K->arrs.size(); a++)
            if (K->arrs[a].space == SP_GLOBAL)
                ki.gid[a] = (int)(std::lower_bound(names.begin(), names.end(), K->arrs[a].name) - names.begin());
        Config cfg;
        cfg.bits = bits; cfg.input_mode = input_mode; cfg.input_range = input_range; cfg.checks = checks;
        if (wmax) cfg.wmax = wmax;
        Results res;
        Slot slots[N_KINDS];
        Exec ex(cfg, ki, *reinterpret_cast<const Launch*>(launch), seed, 0, 0, 0, slots, res);
        /* capture initial contents before running */
        ex.run();
        if (names.size() > max_arrays) throw Error(E_ARG, "too many arrays");
        *n_arrays = (uint32_t)names.size();
        uint64_t off = 0;
        for (size_t g = 0; g < names.size(); g++) {
            size_t a = 0;
            for (; a < K->arrs.size(); a++) if (ki.gid[a] == (int)g) break;
            uint32_t n = ex.size[a];
            sizes[g] = n;
            if (off + n > cap) throw Error(E_ARG, "output buffer too small");
            for (uint32_t i = 0; i < n; i++) {
                init_out[off + i] = ex.init_val((uint32_t)g, i);
                final_out[off + i] = ex.gval[a][i];
            }
            off += n;
        }
        for (int i = 0; i < 16; i++) counts[i] = 0;
        counts[0] = (int64_t)res.instances;
        for (int kind = 0; kind < N_KINDS; kind++) counts[1 + kind] = (int64_t)slots[kind].count;
        return 0;
    } catch (const orc::Error& e) {
        or_err = e.what();
        return e.code;
    } catch (const std::exception& e) {
        or_err = e.what();
        return -1;
    }
}

/* Data-flow relation of one kernel for one launch/seed (H5): one row per
 * in-bounds shared/global read.  Runs in VC-literal mode, so every row has been
 * cross-checked against literal enumeration of all writer threads. */
int or_dataflow(const char* text, const or_launch* launch, uint64_t seed, uint32_t bits, uint32_t* rows,
                uint64_t cap_rows, uint64_t* n_rows) {
    using namespace orc;
    try {
        std::unique_ptr<Kernel> K = parse_kernel(text);
        check_launch(*K, *reinterpret_cast<const Launch*>(launch));
        KInfo ki;
        ki.K = K.get();
        Lowerer lw(ki.prog);
        lw.lower(K->body);
        Ins end; end.k = IN_END;
        ki.prog.ins.push_back(end);
        std::vector<std::string> names;
        for (auto& A : K->arrs) if (A.space == SP_GLOBAL) names.push_back(A.name);
        std::sort(names.begin(), names.end());
        ki.gid.assign(K->arrs.size(), -1);
        for (size_t a = 0; a < K->arrs.size(); a++)
            if (K->arrs[a].space == SP_GLOBAL)
                ki.gid[a] = (int)(std::lower_bound(names.begin(), names.end(), K->arrs[a].name) - names.begin());
        Config cfg;
        cfg.bits = bits; cfg.vcliteral = true; cfg.dataflow = true; cfg.checks = CHK_RACE | CHK_OOB;
        Results res;
        Slot slots[N_KINDS];
        Exec ex(cfg, ki, *reinterpret_cast<const Launch*>(launch), seed, 0, 0, 0, slots, res);
        ex.run();
        *n_rows = res.df.size();
        for (size_t i = 0; i < res.df.size() && i < cap_rows; i++) memcpy(rows + i * 10, &res.df[i], sizeof(DFRow));
        return 0;
    } catch (const orc::Error& e) {
        or_err = e.what();
        return e.code;
    } catch (const std::exception& e) {
        or_err = e.what();
        return -1;
    }
}

/* Lock-step comparison of a pair (X25): for every
 * instance of the space, the first divergence of the kernels' shared contents after
 * rounds < lock_rounds, as rows of 10 words [launch, seed_idx, block, round, array,
 * addr, val_src, val_tgt, written_src, written_tgt] in (launch, seed) order. */
int or_lockstep(const char* src, const char* tgt, const or_space* sp, uint32_t lock_rounds, uint32_t* rows,
                uint64_t cap_rows, uint64_t* n_rows) {
    using namespace orc;
    try {
        if (!src || !tgt || !sp || !n_rows) throw Error(E_ARG, "null argument");
        std::unique_ptr<Kernel> ks = parse_kernel(src), kt = parse_kernel(tgt);
        Space S;
        S.launch_src = reinterpret_cast<const Launch*>(sp->launch_src);
        S.launch_tgt = reinterpret_cast<const Launch*>(sp->launch_tgt);
        S.n_launch = sp->n_launch;
        S.seed_base = sp->seed_base;
        S.n_seeds = sp->n_seeds;
        S.rank = sp->rank;
        S.world = sp->world ? sp->world : 1;
        S.cfg.bits = sp->bits ? sp->bits : 32;
        S.cfg.input_mode = sp->input_mode;
        S.cfg.input_range = sp->input_range;
        S.cfg.checks = sp->checks;
        S.cfg.wmax = sp->wmax ? sp->wmax : 32;
        S.cfg.lock_rounds = lock_rounds;
        S.mode = sp->mode;
        Results res;
        run_space({ks.get(), kt.get()}, {S.launch_src, S.launch_tgt ? S.launch_tgt : S.launch_src}, S, res, false);
        *n_rows = res.div.size();
        for (size_t i = 0; i < res.div.size() && i < cap_rows; i++) memcpy(rows + i * 10, &res.div[i], sizeof(DivRow));
        return 0;
    } catch (const orc::Error& e) {
        or_err = e.what();
        return e.code;
    } catch (const std::exception& e) {
        or_err = e.what();
        return -1;
    }
}

/* PRF test hooks (X8) */
uint64_t or_sm64(uint64_t x) { return orc::sm64(x); }
uint32_t or_rand32(uint64_t seed, uint64_t tag, uint64_t idx) { return orc::rand32(seed, tag, idx); }

}  /* extern "C" */
