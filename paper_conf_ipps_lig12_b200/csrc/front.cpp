// front.cpp — lexer, Pratt parser, scope/type checker and uniformity analysis
// of the kernel IR (product path of libpgvc; independent of oracle/).
#include "front.hpp"

#include <algorithm>
#include <cctype>
#include <cstring>
#include <map>
#include <set>

#include "../../include/pgvc.h"

namespace pgf {

namespace {

std::string where(int line, int col) { return std::to_string(line) + ":" + std::to_string(col) + ": "; }

// ------------------------------------------------------------------ tokens
enum class TT : uint8_t { End, Ident, Int, Punct };

struct Token {
    TT t = TT::End;
    std::string text;
    uint64_t value = 0;
    bool unsigned_suffix = false;
    int line = 1, col = 1;
};

class Lexer {
public:
    explicit Lexer(const std::string& s) : src_(s) {}

    std::vector<Token> run() {
        std::vector<Token> out;
        for (;;) {
            skip_space();
            Token tk;
            tk.line = line_;
            tk.col = col_;
            if (pos_ >= src_.size()) {
                out.push_back(tk);
                return out;
            }
            char c = src_[pos_];
            if (std::isalpha((unsigned char)c) || c == '_') {
                size_t b = pos_;
                while (pos_ < src_.size() && (std::isalnum((unsigned char)src_[pos_]) || src_[pos_] == '_')) bump();
                tk.t = TT::Ident;
                tk.text = src_.substr(b, pos_ - b);
            } else if (std::isdigit((unsigned char)c)) {
                number(tk);
            } else {
                punct(tk);
            }
            out.push_back(tk);
        }
    }

private:
    const std::string& src_;
    size_t pos_ = 0;
    int line_ = 1, col_ = 1;

    void bump() {
        if (src_[pos_] == '\n') {
            line_++;
            col_ = 1;
        } else {
            col_++;
        }
        pos_++;
    }
    [[noreturn]] void fail(const std::string& m) { throw FrontError(PG_E_PARSE, where(line_, col_) + m); }

    void skip_space() {
        for (;;) {
            if (pos_ >= src_.size()) return;
            char c = src_[pos_];
            if (std::isspace((unsigned char)c)) {
                bump();
            } else if (c == '/' && pos_ + 1 < src_.size() && src_[pos_ + 1] == '/') {
                while (pos_ < src_.size() && src_[pos_] != '\n') bump();
            } else if (c == '/' && pos_ + 1 < src_.size() && src_[pos_ + 1] == '*') {
                int l = line_, cc = col_;
                bump();
                bump();
                while (pos_ + 1 < src_.size() && !(src_[pos_] == '*' && src_[pos_ + 1] == '/')) bump();
                if (pos_ + 1 >= src_.size()) throw FrontError(PG_E_PARSE, where(l, cc) + "unterminated comment");
                bump();
                bump();
            } else {
                return;
            }
        }
    }

    void number(Token& tk) {
        uint64_t v = 0;
        size_t b = pos_;
        bool hex = src_[pos_] == '0' && pos_ + 1 < src_.size() && (src_[pos_ + 1] == 'x' || src_[pos_ + 1] == 'X');
        if (hex) {
            bump();
            bump();
            size_t d0 = pos_;
            while (pos_ < src_.size() && std::isxdigit((unsigned char)src_[pos_])) {
                int d = std::isdigit((unsigned char)src_[pos_]) ? src_[pos_] - '0'
                                                                 : std::tolower((unsigned char)src_[pos_]) - 'a' + 10;
                v = v * 16 + (uint64_t)d;
                if (v > 0xFFFFFFFFull) fail("integer literal too large");
                bump();
            }
            if (pos_ == d0) fail("bad hex literal");
        } else {
            while (pos_ < src_.size() && std::isdigit((unsigned char)src_[pos_])) {
                v = v * 10 + (uint64_t)(src_[pos_] - '0');
                if (v > 0xFFFFFFFFull) fail("integer literal too large");
                bump();
            }
        }
        while (pos_ < src_.size() && std::strchr("uUlL", src_[pos_])) {
            if (src_[pos_] == 'u' || src_[pos_] == 'U') tk.unsigned_suffix = true;
            bump();
        }
        if (pos_ < src_.size() && (std::isalnum((unsigned char)src_[pos_]) || src_[pos_] == '_'))
            fail("bad integer literal");
        tk.t = TT::Int;
        tk.value = v;
        tk.text = src_.substr(b, pos_ - b);
    }

    void punct(Token& tk) {
        static const char* multi[] = {"<<=", ">>=", "<<", ">>", "<=", ">=", "==", "!=", "&&", "||", "++", "--",
                                      "+=",  "-=",  "*=", "/=", "%=", "&=", "|=", "^=", nullptr};
        for (int i = 0; multi[i]; i++) {
            size_t n = std::strlen(multi[i]);
            if (src_.compare(pos_, n, multi[i]) == 0) {
                tk.t = TT::Punct;
                tk.text = multi[i];
                for (size_t k = 0; k < n; k++) bump();
                return;
            }
        }
        char c = src_[pos_];
        if (!std::strchr("+-*/%<>=!~&|^?:;,.()[]{}", c)) fail(std::string("unexpected character '") + c + "'");
        tk.t = TT::Punct;
        tk.text = std::string(1, c);
        bump();
    }
};

// ------------------------------------------------------------------ parser
const char* const kKeywords[] = {"int",    "unsigned", "kernel", "global",   "shared",   "__shared__", "if",
                                 "else",   "for",      "while",  "sync",     "__syncthreads", "return", "break",
                                 "continue", "in",     "out",    "inout",    "min",      "max",        "tid",
                                 "bid",    "bdim",     "gdim",   "threadIdx", "blockIdx", "blockDim",  "gridDim",
                                 nullptr};

bool is_keyword(const std::string& s) {
    for (int i = 0; kKeywords[i]; i++)
        if (s == kKeywords[i]) return true;
    return false;
}

int builtin_group(const std::string& s) {
    if (s == "tid" || s == "threadIdx") return 0;
    if (s == "bid" || s == "blockIdx") return 3;
    if (s == "bdim" || s == "blockDim") return 6;
    if (s == "gdim" || s == "gridDim") return 9;
    return -1;
}

Ty arith(Ty a, Ty b) { return (a == Ty::U32 || b == Ty::U32) ? Ty::U32 : Ty::I32; }

struct BinInfo {
    const char* tok;
    int prec;
    Bop op;
};
// precedence climbing table (C): | 6, ^ 7, & 8, == != 9, relational 10, shifts 11, additive 12, multiplicative 13
const BinInfo kBin[] = {{"|", 6, Bop::Or},   {"^", 7, Bop::Xor},  {"&", 8, Bop::And},  {"==", 9, Bop::Eq},
                        {"!=", 9, Bop::Ne},  {"<", 10, Bop::Lt},  {"<=", 10, Bop::Le}, {">", 10, Bop::Gt},
                        {">=", 10, Bop::Ge}, {"<<", 11, Bop::Shl}, {">>", 11, Bop::Shr}, {"+", 12, Bop::Add},
                        {"-", 12, Bop::Sub}, {"*", 13, Bop::Mul}, {"/", 13, Bop::Div}, {"%", 13, Bop::Rem}};

class Parser {
public:
    Parser(const std::string& text, Kernel& k) : toks_(Lexer(text).run()), K(k) {}

    void parse() {
        expect_kw("kernel");
        K.name = ident("kernel name");
        params();
        expect("{");
        scopes_.emplace_back();
        std::vector<Stmt*> top;
        while (!at("}")) {
            if (peek().t == TT::End) fail("unexpected end of input");
            if (at_kw("shared") || at_kw("__shared__")) {
                shared_decl();
                continue;
            }
            top.push_back(statement());
        }
        next();
        scopes_.pop_back();
        scopes_.pop_back();
        if (peek().t != TT::End) fail("trailing input after kernel");
        K.body = seq(std::move(top), toks_[0]);
    }

private:
    std::vector<Token> toks_;
    size_t p_ = 0;
    Kernel& K;
    std::vector<std::map<std::string, int>> scopes_;
    std::map<std::string, int> arrays_;
    std::vector<int> loops_;
    int hidden_ = 0;

    const Token& peek(size_t k = 0) const { return toks_[std::min(p_ + k, toks_.size() - 1)]; }
    const Token& next() { return toks_[p_ < toks_.size() - 1 ? p_++ : p_]; }
    bool at(const char* s) const { return peek().t == TT::Punct && peek().text == s; }
    bool at_kw(const char* s) const { return peek().t == TT::Ident && peek().text == s; }
    [[noreturn]] void fail(const std::string& m) const {
        throw FrontError(PG_E_PARSE, where(peek().line, peek().col) + m);
    }
    [[noreturn]] static void type_error(const Token& t, const std::string& m) {
        throw FrontError(PG_E_TYPE, where(t.line, t.col) + m);
    }
    void expect(const char* s) {
        if (!at(s)) fail(std::string("expected '") + s + "'");
        next();
    }
    void expect_kw(const char* s) {
        if (!at_kw(s)) fail(std::string("expected '") + s + "'");
        next();
    }
    std::string ident(const char* what) {
        if (peek().t != TT::Ident) fail(std::string("expected ") + what);
        return next().text;
    }

    Node* node(NK k, const Token& t) {
        K.node_pool.emplace_back(new Node());
        Node* n = K.node_pool.back().get();
        n->kind = k;
        n->line = t.line;
        n->col = t.col;
        return n;
    }
    Stmt* stmt(SK k, const Token& t) {
        K.stmt_pool.emplace_back(new Stmt());
        Stmt* s = K.stmt_pool.back().get();
        s->kind = k;
        s->line = t.line;
        s->col = t.col;
        return s;
    }
    Stmt* seq(std::vector<Stmt*> v, const Token& t) {
        Stmt* s = stmt(SK::Seq, t);
        s->seq = std::move(v);
        return s;
    }
    int site(int arr, bool store) {
        K.sites.push_back(SiteInfo{arr, store});
        return (int)K.sites.size() - 1;
    }

    bool at_type() const { return at_kw("int") || at_kw("unsigned"); }
    Ty type() {
        if (at_kw("int")) {
            next();
            return Ty::I32;
        }
        if (at_kw("unsigned")) {
            next();
            if (at_kw("int")) next();
            return Ty::U32;
        }
        fail("expected a type");
    }

    int find_var(const std::string& n) const {
        for (auto it = scopes_.rbegin(); it != scopes_.rend(); ++it) {
            auto f = it->find(n);
            if (f != it->end()) return f->second;
        }
        return -1;
    }
    int new_var(const std::string& n, Ty ty, const Token& t) {
        if (is_keyword(n)) type_error(t, "reserved name '" + n + "'");
        if (scopes_.back().count(n) || arrays_.count(n)) type_error(t, "redeclaration of '" + n + "'");
        VarDecl v;
        v.name = n;
        v.ty = ty;
        K.vars.push_back(v);
        scopes_.back()[n] = (int)K.vars.size() - 1;
        return (int)K.vars.size() - 1;
    }
    int hidden_var(Ty ty) {
        VarDecl v;
        v.name = "__h" + std::to_string(hidden_++);
        v.ty = ty;
        v.hidden = true;
        K.vars.push_back(v);
        return (int)K.vars.size() - 1;
    }
    int add_array(ArrayDecl a, const Token& t) {
        if (is_keyword(a.name) || arrays_.count(a.name) || find_var(a.name) >= 0)
            type_error(t, "bad or duplicate array name '" + a.name + "'");
        a.slot = K.n_space(a.space);
        K.arrays.push_back(a);
        arrays_[a.name] = (int)K.arrays.size() - 1;
        return (int)K.arrays.size() - 1;
    }

    // --- kernel signature: global arrays and scalars; sizes parsed after the list
    void params() {
        expect("(");
        scopes_.emplace_back();
        std::vector<std::pair<int, size_t>> deferred;
        if (!at(")")) {
            for (;;) {
                if (at_kw("global")) {
                    next();
                    ArrayDecl a;
                    a.space = GLOBAL;
                    if (at_kw("in")) a.mode = IN;
                    else if (at_kw("out")) a.mode = OUT;
                    else if (at_kw("inout")) a.mode = INOUT;
                    else fail("expected in, out or inout");
                    next();
                    a.ety = type();
                    Token nt = peek();
                    a.name = ident("array name");
                    expect("[");
                    size_t start = p_;
                    for (int depth = 1; depth > 0;) {
                        if (peek().t == TT::End) fail("unterminated array size");
                        if (at("[")) depth++;
                        if (at("]")) depth--;
                        next();
                    }
                    deferred.push_back({add_array(a, nt), start});
                } else if (at_type()) {
                    Ty ty = type();
                    Token nt = peek();
                    int v = new_var(ident("parameter name"), ty, nt);
                    K.vars[(size_t)v].scalar = true;
                    K.vars[(size_t)v].scalar_index = (int)K.scalars.size();
                    K.scalars.push_back(v);
                } else {
                    fail("expected parameter");
                }
                if (!at(",")) break;
                next();
            }
        }
        expect(")");
        size_t resume = p_;
        for (auto& d : deferred) {
            p_ = d.second;
            size_t s0 = K.sites.size();
            Node* e = expr();
            if (K.sites.size() != s0) type_error(toks_[d.second], "array size may not read memory");
            K.arrays[(size_t)d.first].dims.push_back(e);
            expect("]");
        }
        p_ = resume;
        if (K.scalars.size() > 8) fail("at most 8 scalar parameters");
    }

    void shared_decl() {
        next();
        ArrayDecl a;
        a.space = SHARED;
        a.ety = type();
        Token nt = peek();
        a.name = ident("array name");
        size_t s0 = K.sites.size();
        while (at("[")) {
            next();
            a.dims.push_back(expr());
            expect("]");
        }
        if (a.dims.empty()) fail("shared array needs dimensions");
        if (K.sites.size() != s0) type_error(nt, "array dimension may not read memory");
        add_array(a, nt);
        expect(";");
    }

    // --- expressions (precedence climbing)
    Node* expr() { return ternary(); }

    Node* ternary() {
        Node* c = logic_or();
        if (!at("?")) return c;
        Token t = next();
        Node* a = expr();
        expect(":");
        Node* b = ternary();
        Node* n = node(NK::Select, t);
        n->kids = {c, a, b};
        n->ty = n->opty = arith(a->ty, b->ty);
        return n;
    }
    Node* logic_or() {
        Node* l = logic_and();
        while (at("||")) {
            Token t = next();
            Node* n = node(NK::LOr, t);
            n->kids = {l, logic_and()};
            n->ty = Ty::I32;
            l = n;
        }
        return l;
    }
    Node* logic_and() {
        Node* l = binary(6);
        while (at("&&")) {
            Token t = next();
            Node* n = node(NK::LAnd, t);
            n->kids = {l, binary(6)};
            n->ty = Ty::I32;
            l = n;
        }
        return l;
    }
    const BinInfo* bin_at() const {
        if (peek().t != TT::Punct) return nullptr;
        for (const BinInfo& b : kBin)
            if (peek().text == b.tok) return &b;
        return nullptr;
    }
    Node* make_bin(Bop op, Node* l, Node* r, const Token& t) {
        Node* n = node(NK::Bin, t);
        n->op = op;
        n->kids = {l, r};
        if (op == Bop::Shl || op == Bop::Shr) {
            n->ty = n->opty = l->ty;
        } else if (op >= Bop::Lt) {
            n->opty = arith(l->ty, r->ty);
            n->ty = Ty::I32;
        } else {
            n->ty = n->opty = arith(l->ty, r->ty);
        }
        return n;
    }
    Node* binary(int min_prec) {
        Node* l = unary();
        for (;;) {
            const BinInfo* b = bin_at();
            if (!b || b->prec < min_prec) return l;
            Token t = next();
            Node* r = binary(b->prec + 1);
            l = make_bin(b->op, l, r, t);
        }
    }
    Node* unary() {
        Token t = peek();
        if (at("-") || at("~") || at("!")) {
            next();
            Node* a = unary();
            NK k = t.text == "-" ? NK::Neg : t.text == "~" ? NK::BitNot : NK::LogNot;
            Node* n = node(k, t);
            n->kids = {a};
            n->ty = k == NK::LogNot ? Ty::I32 : a->ty;
            return n;
        }
        if (at("+")) {
            next();
            return unary();
        }
        if (at("(") && peek(1).t == TT::Ident && (peek(1).text == "int" || peek(1).text == "unsigned")) {
            next();
            Ty ty = type();
            expect(")");
            Node* n = node(NK::Cast, t);
            n->kids = {unary()};
            n->ty = ty;
            return n;
        }
        return primary();
    }
    void indices(int arr, std::vector<Node*>& out) {
        const ArrayDecl& a = K.arrays[(size_t)arr];
        size_t rank = a.space == GLOBAL ? 1 : a.dims.size();
        for (size_t d = 0; d < rank; d++) {
            expect("[");
            out.push_back(expr());
            expect("]");
        }
        if (at("[")) fail("too many indices for array '" + a.name + "'");
    }
    Node* primary() {
        Token t = peek();
        if (t.t == TT::Int) {
            next();
            Node* n = node(NK::Lit, t);
            n->lit = (uint32_t)t.value;
            n->ty = (t.unsigned_suffix || t.value > 0x7FFFFFFFull) ? Ty::U32 : Ty::I32;
            return n;
        }
        if (at("(")) {
            next();
            Node* e = expr();
            expect(")");
            return e;
        }
        if (t.t != TT::Ident) fail("expected expression");
        next();
        if (t.text == "min" || t.text == "max") {
            expect("(");
            Node* a = expr();
            expect(",");
            Node* b = expr();
            expect(")");
            Node* n = node(t.text == "min" ? NK::Min : NK::Max, t);
            n->kids = {a, b};
            n->ty = n->opty = arith(a->ty, b->ty);
            return n;
        }
        int g = builtin_group(t.text);
        if (g >= 0) {
            expect(".");
            std::string f = ident("component");
            int c = f == "x" ? 0 : f == "y" ? 1 : f == "z" ? 2 : -1;
            if (c < 0) fail("expected .x, .y or .z");
            Node* n = node(NK::Builtin, t);
            n->ref = g + c;
            n->ty = Ty::U32;  // CUDA uint3 (X2)
            return n;
        }
        auto ai = arrays_.find(t.text);
        if (ai != arrays_.end()) {
            Node* n = node(NK::Elem, t);
            n->ref = ai->second;
            indices(n->ref, n->kids);
            n->site = site(n->ref, false);
            n->ty = K.arrays[(size_t)n->ref].ety;
            K.arrays[(size_t)n->ref].read = true;
            return n;
        }
        int v = find_var(t.text);
        if (v < 0) type_error(t, "undeclared identifier '" + t.text + "'");
        Node* n = node(NK::Var, t);
        n->ref = v;
        n->ty = K.vars[(size_t)v].ty;
        return n;
    }

    // --- statements
    Node* var_ref(int v, const Token& t) {
        Node* n = node(NK::Var, t);
        n->ref = v;
        n->ty = K.vars[(size_t)v].ty;
        return n;
    }
    Node* one(const Token& t) {
        Node* n = node(NK::Lit, t);
        n->lit = 1;
        return n;
    }
    static int compound(const std::string& s, Bop& op) {
        static const char* names[] = {"+=", "-=", "*=", "/=", "%=", "<<=", ">>=", "&=", "|=", "^="};
        static const Bop ops[] = {Bop::Add, Bop::Sub, Bop::Mul, Bop::Div, Bop::Rem,
                                  Bop::Shl, Bop::Shr, Bop::And, Bop::Or,  Bop::Xor};
        for (int i = 0; i < 10; i++)
            if (s == names[i]) {
                op = ops[i];
                return 1;
            }
        return 0;
    }
    // assignment, compound assignment, ++/-- (prefix or postfix); no ';'
    Stmt* assignment() {
        Token t0 = peek();
        int pre = 0;
        if (at("++")) pre = 1;
        if (at("--")) pre = -1;
        if (pre) next();
        Token nt = peek();
        std::string name = ident("assignment target");
        Bop op = Bop::Add;
        auto ai = arrays_.find(name);
        if (ai != arrays_.end()) {
            int arr = ai->second;
            std::vector<Node*> idx;
            indices(arr, idx);
            int first = site(arr, true);
            bool plain = false;
            Node* rhs = nullptr;
            if (pre) {
                op = pre > 0 ? Bop::Add : Bop::Sub;
                rhs = one(t0);
            } else if (at("=")) {
                next();
                plain = true;
            } else if (at("++") || at("--")) {
                op = at("++") ? Bop::Add : Bop::Sub;
                next();
                rhs = one(t0);
            } else if (peek().t == TT::Punct && compound(peek().text, op)) {
                next();
            } else {
                fail("expected assignment");
            }
            K.arrays[(size_t)arr].written = true;
            if (plain) {
                Stmt* s = stmt(SK::Store, nt);
                s->arr = arr;
                s->index = idx;
                s->site = first;
                s->value = expr();
                return s;
            }
            // compound: `first` is the read site, a second site is the write (X21)
            K.sites[(size_t)first].store = false;
            K.arrays[(size_t)arr].read = true;
            int wsite = site(arr, true);
            if (!rhs) rhs = expr();
            std::vector<Stmt*> parts;
            std::vector<Node*> tidx;
            for (Node* e : idx) {
                int h = hidden_var(e->ty);
                Stmt* as = stmt(SK::Assign, nt);
                as->var = h;
                as->value = e;
                parts.push_back(as);
                tidx.push_back(var_ref(h, nt));
            }
            Node* ld = node(NK::Elem, nt);
            ld->ref = arr;
            ld->kids = tidx;
            ld->site = first;
            ld->ty = K.arrays[(size_t)arr].ety;
            Stmt* st = stmt(SK::Store, nt);
            st->arr = arr;
            st->index = tidx;
            st->site = wsite;
            st->value = make_bin(op, ld, rhs, nt);
            parts.push_back(st);
            return seq(std::move(parts), nt);
        }
        int v = find_var(name);
        if (v < 0) type_error(nt, "undeclared identifier '" + name + "'");
        Stmt* s = stmt(SK::Assign, nt);
        s->var = v;
        Node* rhs = nullptr;
        if (pre) {
            op = pre > 0 ? Bop::Add : Bop::Sub;
            rhs = one(t0);
        } else if (at("=")) {
            next();
            s->value = expr();
            return s;
        } else if (at("++") || at("--")) {
            op = at("++") ? Bop::Add : Bop::Sub;
            next();
            rhs = one(t0);
        } else if (peek().t == TT::Punct && compound(peek().text, op)) {
            next();
            rhs = expr();
        } else {
            fail("expected assignment");
        }
        s->value = make_bin(op, var_ref(v, nt), rhs, nt);
        return s;
    }
    Stmt* declaration() {
        Token t0 = peek();
        Ty ty = type();
        std::vector<Stmt*> parts;
        for (;;) {
            Token nt = peek();
            std::string name = ident("variable name");
            if (at("[")) {
                if (is_keyword(name) || scopes_.back().count(name) || arrays_.count(name) || find_var(name) >= 0)
                    type_error(nt, "redeclaration of '" + name + "'");
                ArrayDecl a;
                a.name = name;
                a.space = PRIVATE;
                a.ety = ty;
                while (at("[")) {
                    next();
                    if (peek().t != TT::Int) fail("private array dimension must be an integer literal");
                    Node* d = node(NK::Lit, peek());
                    d->lit = (uint32_t)next().value;
                    a.dims.push_back(d);
                    expect("]");
                }
                int id = add_array(a, nt);
                Stmt* s = stmt(SK::PrivDecl, nt);
                s->arr = id;
                parts.push_back(s);
            } else {
                Node* init = nullptr;
                if (at("=")) {
                    next();
                    init = expr();
                }
                Stmt* s = stmt(SK::Assign, nt);
                s->var = new_var(name, ty, nt);  // after its initialiser (C scope rule)
                if (!init) {
                    init = node(NK::Lit, nt);  // X21: uninitialised locals are 0
                }
                s->value = init;
                parts.push_back(s);
            }
            if (!at(",")) break;
            next();
        }
        return parts.size() == 1 ? parts[0] : seq(std::move(parts), t0);
    }
    Stmt* scoped_statement() {
        scopes_.emplace_back();
        Stmt* s = statement();
        scopes_.pop_back();
        return s;
    }
    Stmt* statement() {
        Token t = peek();
        if (at("{")) {
            next();
            scopes_.emplace_back();
            std::vector<Stmt*> v;
            while (!at("}")) {
                if (peek().t == TT::End) fail("unexpected end of input");
                v.push_back(statement());
            }
            next();
            scopes_.pop_back();
            return seq(std::move(v), t);
        }
        if (at(";")) {
            next();
            return stmt(SK::Nop, t);
        }
        if (at_kw("shared") || at_kw("__shared__")) fail("shared declarations must be at the top level of the kernel body");
        if (at_type()) {
            Stmt* s = declaration();
            expect(";");
            return s;
        }
        if (at_kw("if")) {
            next();
            expect("(");
            Stmt* s = stmt(SK::If, t);
            s->cond = expr();
            expect(")");
            s->body = scoped_statement();
            if (at_kw("else")) {
                next();
                s->other = scoped_statement();
            }
            return s;
        }
        if (at_kw("for")) {
            next();
            Stmt* s = stmt(SK::Loop, t);
            s->loop = K.n_loops++;
            scopes_.emplace_back();
            expect("(");
            if (!at(";")) s->init = at_type() ? declaration() : assignment();
            expect(";");
            loops_.push_back(s->loop);
            if (!at(";")) s->cond = expr();
            expect(";");
            if (!at(")")) s->step = assignment();
            expect(")");
            s->body = scoped_statement();
            loops_.pop_back();
            scopes_.pop_back();
            return s;
        }
        if (at_kw("while")) {
            next();
            Stmt* s = stmt(SK::Loop, t);
            s->loop = K.n_loops++;
            loops_.push_back(s->loop);
            expect("(");
            s->cond = expr();
            expect(")");
            s->body = scoped_statement();
            loops_.pop_back();
            return s;
        }
        if (at_kw("sync") || at_kw("__syncthreads")) {
            bool cuda = at_kw("__syncthreads");
            next();
            if (cuda) {
                expect("(");
                expect(")");
            }
            expect(";");
            Stmt* s = stmt(SK::Sync, t);
            s->site = site(-1, false);
            s->has_sync = true;
            K.n_syncs++;
            return s;
        }
        if (at_kw("return")) {
            next();
            expect(";");
            return stmt(SK::Return, t);
        }
        if (at_kw("break") || at_kw("continue")) {
            bool brk = at_kw("break");
            next();
            expect(";");
            if (loops_.empty()) type_error(t, std::string(brk ? "break" : "continue") + " outside a loop");
            Stmt* s = stmt(brk ? SK::Break : SK::Continue, t);
            s->loop = loops_.back();
            return s;
        }
        Stmt* s = assignment();
        expect(";");
        return s;
    }
};

// ------------------------------------------------------------------ uniformity analysis
// A value is block-uniform when it depends only on literals, scalar parameters,
// bid/bdim/gdim and uniform variables (never on tid or on memory).  Control
// flow on uniform conditions is taken identically by every thread of the
// block; only there may a barrier appear (X18).
class Uniformity {
public:
    explicit Uniformity(Kernel& k) : K(k), loop_nonuniform_jump_(std::max(1, k.n_loops), false) {}

    void run() {
        do {
            changed_ = false;
            walk(K.body, true);
        } while (changed_);
        mark_nodes(K.body);
        check_syncs(K.body, true);
        // grid uniformity: variables whose uniform value never depends on bid
        grid_.assign(K.vars.size(), true);
        for (size_t v = 0; v < K.vars.size(); v++) grid_[v] = K.vars[v].uniform;
        do {
            changed_ = false;
            grid_walk(K.body);
        } while (changed_);
        K.grid_uniform_control = grid_control(K.body) && !K.div_barrier;
    }

private:
    Kernel& K;
    std::vector<bool> loop_nonuniform_jump_;
    std::vector<bool> grid_;
    bool changed_ = false;

    bool grid_uniform(const Node* n) const {
        switch (n->kind) {
        case NK::Lit: return true;
        case NK::Var: return grid_[(size_t)n->ref];
        case NK::Builtin: return n->ref >= 6;  // bdim, gdim
        case NK::Elem: return false;
        default:
            for (const Node* c : n->kids)
                if (!grid_uniform(c)) return false;
            return true;
        }
    }
    void grid_walk(const Stmt* s) {
        if (!s) return;
        if (s->kind == SK::Assign && grid_[(size_t)s->var] && !grid_uniform(s->value)) {
            grid_[(size_t)s->var] = false;
            changed_ = true;
        }
        for (const Stmt* c : s->seq) grid_walk(c);
        grid_walk(s->body);
        grid_walk(s->other);
        grid_walk(s->init);
        grid_walk(s->step);
    }
    bool grid_control(const Stmt* s) const {
        if (!s) return true;
        if ((s->kind == SK::If || s->kind == SK::Loop) && s->uniform && s->cond && !grid_uniform(s->cond)) return false;
        for (const Stmt* c : s->seq)
            if (!grid_control(c)) return false;
        return grid_control(s->body) && grid_control(s->other) && grid_control(s->init) && grid_control(s->step);
    }

    bool uniform(const Node* n) const {
        switch (n->kind) {
        case NK::Lit: return true;
        case NK::Var: return K.vars[(size_t)n->ref].uniform;
        case NK::Builtin: return n->ref >= 3;
        case NK::Elem: return false;
        default:
            for (const Node* c : n->kids)
                if (!uniform(c)) return false;
            return true;
        }
    }
    void demote(int v) {
        if (K.vars[(size_t)v].uniform) {
            K.vars[(size_t)v].uniform = false;
            changed_ = true;
        }
    }
    bool walk(Stmt* s, bool u) {  // returns has_sync
        if (!s) return false;
        bool sy = false;
        switch (s->kind) {
        case SK::Seq:
            for (Stmt* c : s->seq) sy |= walk(c, u);
            break;
        case SK::Assign:
            if (!u || !uniform(s->value)) demote(s->var);
            break;
        case SK::If: {
            bool cu = u && uniform(s->cond);
            s->uniform = cu;
            sy |= walk(s->body, cu);
            sy |= walk(s->other, cu);
            break;
        }
        case SK::Loop: {
            sy |= walk(s->init, u);
            bool lu = u && (!s->cond || uniform(s->cond)) && !loop_nonuniform_jump_[(size_t)s->loop];
            s->uniform = lu;
            sy |= walk(s->body, lu);
            sy |= walk(s->step, lu);
            break;
        }
        case SK::Break:
        case SK::Continue:
            s->uniform = u;
            if (!u && !loop_nonuniform_jump_[(size_t)s->loop]) {
                loop_nonuniform_jump_[(size_t)s->loop] = true;
                changed_ = true;
            }
            break;
        case SK::Return:
            s->uniform = u;
            break;
        case SK::Sync:
            sy = true;
            break;
        default:
            break;
        }
        s->has_sync = sy;
        return sy;
    }
    void mark(Node* n) {
        if (!n) return;
        for (Node* c : n->kids) mark(c);
        n->uniform = uniform(n);
    }
    void mark_nodes(Stmt* s) {
        if (!s) return;
        for (Stmt* c : s->seq) mark_nodes(c);
        mark(s->value);
        mark(s->cond);
        for (Node* i : s->index) mark(i);
        mark_nodes(s->body);
        mark_nodes(s->other);
        mark_nodes(s->init);
        mark_nodes(s->step);
    }
    void check_syncs(const Stmt* s, bool u) {
        if (!s) return;
        switch (s->kind) {
        case SK::Sync:
            if (!u) K.div_barrier = true;   // checked at run time (X18)
            break;
        case SK::Seq:
            for (const Stmt* c : s->seq) check_syncs(c, u);
            break;
        case SK::If:
            check_syncs(s->body, u && s->uniform);
            check_syncs(s->other, u && s->uniform);
            break;
        case SK::Loop:
            check_syncs(s->init, u);
            check_syncs(s->body, u && s->uniform);
            check_syncs(s->step, u && s->uniform);
            break;
        default:
            break;
        }
    }
};

// 32-bit launch-time arithmetic (X2 at w = 32)
uint32_t binop32(Bop op, Ty ty, uint32_t a, uint32_t b) {
    int32_t x = (int32_t)a, y = (int32_t)b;
    bool s = ty == Ty::I32;
    switch (op) {
    case Bop::Add: return a + b;
    case Bop::Sub: return a - b;
    case Bop::Mul: return a * b;
    case Bop::Div:
        if (!s) return b ? a / b : 0xFFFFFFFFu;
        if (y == 0) return x < 0 ? 1u : 0xFFFFFFFFu;
        if (x == INT32_MIN && y == -1) return a;
        return (uint32_t)(x / y);
    case Bop::Rem:
        if (!s) return b ? a % b : a;
        if (y == 0) return a;
        if (y == -1) return 0;
        return (uint32_t)(x % y);
    case Bop::Shl: return b >= 32 ? 0u : a << b;
    case Bop::Shr:
        if (!s) return b >= 32 ? 0u : a >> b;
        return b >= 32 ? (x < 0 ? 0xFFFFFFFFu : 0u) : (uint32_t)(x >> b);
    case Bop::And: return a & b;
    case Bop::Or: return a | b;
    case Bop::Xor: return a ^ b;
    case Bop::Lt: return s ? x < y : a < b;
    case Bop::Le: return s ? x <= y : a <= b;
    case Bop::Gt: return s ? x > y : a > b;
    case Bop::Ge: return s ? x >= y : a >= b;
    case Bop::Eq: return a == b;
    case Bop::Ne: return a != b;
    }
    return 0;
}

}  // namespace

std::unique_ptr<Kernel> parse_kernel(const std::string& text) {
    std::unique_ptr<Kernel> k(new Kernel());
    Parser p(text, *k);
    p.parse();
    Uniformity(*k).run();
    if (k->sites.size() > 0xFFFE) throw FrontError(PG_E_LIMIT, "too many access sites");
    if (k->n_space(GLOBAL) > 16 || k->n_space(SHARED) > 16 || k->n_space(PRIVATE) > 16)
        throw FrontError(PG_E_LIMIT, "at most 16 arrays per space");
    return k;
}

uint32_t eval_launch_expr(const Kernel& k, const Node* e, const uint32_t gdim[3], const uint32_t bdim[3],
                          const int32_t* scalars) {
    auto ev = [&](auto&& self, const Node* n) -> uint32_t {
        switch (n->kind) {
        case NK::Lit: return n->lit;
        case NK::Var: {
            const VarDecl& v = k.vars[(size_t)n->ref];
            if (!v.scalar)
                throw FrontError(PG_E_TYPE, where(n->line, n->col) + "size expression may only use scalars, bdim, gdim");
            return (uint32_t)scalars[v.scalar_index];
        }
        case NK::Builtin:
            if (n->ref >= 6 && n->ref < 9) return bdim[n->ref - 6];
            if (n->ref >= 9) return gdim[n->ref - 9];
            throw FrontError(PG_E_TYPE, where(n->line, n->col) + "size expression may only use scalars, bdim, gdim");
        case NK::Elem:
            throw FrontError(PG_E_TYPE, where(n->line, n->col) + "size expression may not read memory");
        case NK::Neg: return 0u - self(self, n->kids[0]);
        case NK::BitNot: return ~self(self, n->kids[0]);
        case NK::LogNot: return self(self, n->kids[0]) == 0;
        case NK::Cast: return self(self, n->kids[0]);
        case NK::LAnd: return self(self, n->kids[0]) ? (self(self, n->kids[1]) != 0) : 0u;
        case NK::LOr: return self(self, n->kids[0]) ? 1u : (self(self, n->kids[1]) != 0);
        case NK::Select: return self(self, n->kids[0]) ? self(self, n->kids[1]) : self(self, n->kids[2]);
        case NK::Min:
        case NK::Max: {
            uint32_t a = self(self, n->kids[0]), b = self(self, n->kids[1]);
            bool lt = binop32(Bop::Lt, n->opty, a, b) != 0;
            return (n->kind == NK::Min) == lt ? a : b;
        }
        case NK::Bin: return binop32(n->op, n->opty, self(self, n->kids[0]), self(self, n->kids[1]));
        }
        return 0;
    };
    return ev(ev, e);
}

}  // namespace pgf
