// front.hpp — IR front end of libpgvc (product path): AST of the kernel IR,
// parser, scope/type checking and the uniformity analysis that decides which
// control flow is block-uniform (real branches, barriers allowed) and which
// is thread-dependent (if-converted, barrier-free).  DESIGN.md §4.
//
// The IR is the C subset the paper's kernels are written in (PAPER.md
// L122-L171, L331-L374, L392-L399, L723-L727, L825-L837).
#pragma once
#include <cstdint>
#include <memory>
#include <stdexcept>
#include <string>
#include <vector>

namespace pgf {

struct FrontError : std::runtime_error {
    int status;  // PG_E_PARSE / PG_E_TYPE / PG_E_LIMIT
    FrontError(int s, const std::string& m) : std::runtime_error(m), status(s) {}
};

enum class Ty : uint8_t { I32, U32 };

enum class Bop : uint8_t { Add, Sub, Mul, Div, Rem, Shl, Shr, And, Or, Xor, Lt, Le, Gt, Ge, Eq, Ne };

enum class NK : uint8_t { Lit, Var, Builtin, Elem, Neg, BitNot, LogNot, Bin, LAnd, LOr, Select, Min, Max, Cast };

// builtin ids: 0..2 tid.xyz, 3..5 bid.xyz, 6..8 bdim.xyz, 9..11 gdim.xyz
struct Node {
    NK kind = NK::Lit;
    Ty ty = Ty::I32;     // result type
    Ty opty = Ty::I32;   // operation type (usual arithmetic conversions; shift: left type)
    Bop op = Bop::Add;
    uint32_t lit = 0;
    int ref = -1;        // var id, builtin id or array id
    int site = -1;       // access site (Elem)
    std::vector<Node*> kids;  // operands (Bin/LAnd/LOr: 2, Select: 3) or indices (Elem)
    bool uniform = false;     // set by the uniformity analysis
    int line = 0, col = 0;
};

enum class SK : uint8_t { Seq, Assign, Store, PrivDecl, If, Loop, Sync, Return, Break, Continue, Nop };

struct Stmt {
    SK kind = SK::Nop;
    std::vector<Stmt*> seq;   // Seq
    int var = -1;             // Assign
    int arr = -1;             // Store / PrivDecl
    std::vector<Node*> index; // Store
    Node* value = nullptr;    // Assign / Store value
    Node* cond = nullptr;     // If / Loop (nullptr loop cond = true)
    Stmt* body = nullptr;     // If-then / Loop body
    Stmt* other = nullptr;    // If-else
    Stmt* init = nullptr;     // Loop (for) init, runs before the loop
    Stmt* step = nullptr;     // Loop (for) step
    int site = -1;            // Store / Sync
    int loop = -1;            // Loop id; Break/Continue: target loop id
    bool uniform = false;     // If/Loop: block-uniform control; Return/Break/Continue: taken uniformly
    bool has_sync = false;    // contains a barrier (If/Loop/Seq)
    int line = 0, col = 0;
};

enum Space : uint8_t { GLOBAL = 0, SHARED = 1, PRIVATE = 2 };
enum Mode : uint8_t { IN = 0, OUT = 1, INOUT = 2 };

struct ArrayDecl {
    std::string name;
    Space space = GLOBAL;
    Ty ety = Ty::I32;
    Mode mode = IN;
    std::vector<Node*> dims;  // GLOBAL: one flat size; SHARED: dims (uniform); PRIVATE: literal dims
    int slot = 0;             // index among arrays of its space, declaration order
    bool written = false;     // some store site targets it
    bool read = false;        // some load site reads it
};

struct VarDecl {
    std::string name;
    Ty ty = Ty::I32;
    bool scalar = false;  // kernel scalar parameter
    int scalar_index = -1;
    bool uniform = true;  // analysis result
    bool hidden = false;
};

struct SiteInfo {
    int arr = -1;        // -1 for a sync site
    bool store = false;
};

struct Kernel {
    std::string name;
    std::vector<VarDecl> vars;
    std::vector<ArrayDecl> arrays;
    std::vector<int> scalars;  // var ids of scalar params, in order
    std::vector<SiteInfo> sites;
    int n_loops = 0;
    int n_syncs = 0;
    // every block-uniform branch / loop condition is also grid-uniform (does not
    // depend on bid): emulated blocks with different bid share one round structure
    // and can run lock-step in one CTA
    bool grid_uniform_control = true;
    // some `sync` sits under thread-dependent control flow: threads of a block may wait at
    // different barriers, which the run-time check X18 reports (BARRIER_DIV).  Such kernels
    // are compiled with per-thread branches and per-thread resume points (codegen.cpp)
    bool div_barrier = false;
    Stmt* body = nullptr;
    std::vector<std::unique_ptr<Node>> node_pool;
    std::vector<std::unique_ptr<Stmt>> stmt_pool;

    int n_space(Space s) const {
        int n = 0;
        for (auto& a : arrays) n += a.space == s;
        return n;
    }
};

// Parse + check one kernel.  Throws FrontError.
std::unique_ptr<Kernel> parse_kernel(const std::string& text);

// Evaluate a uniform launch-time expression (array sizes / shared dims) with
// 32-bit arithmetic: may reference scalars, bdim.*, gdim.* and literals.
uint32_t eval_launch_expr(const Kernel& k, const Node* e, const uint32_t gdim[3], const uint32_t bdim[3],
                          const int32_t* scalars);

// Generate the CUDA C++ source of the evaluation kernel (codegen.cpp).
struct CodegenOptions {
    uint32_t bits = 32;
    uint32_t checks = 0;
    uint32_t bank_model = 0;
    uint32_t wmax = 32;
    bool fast = false;   // optimistic pass: in-place commits, race detection only
    uint32_t ms = 1;     // optimistic pass of a seed-oblivious kernel: seeds per lane
};
std::string generate_cuda(const Kernel& k, const CodegenOptions& opt);

// Multi-seed lanes: true when no address, access guard, branch or loop condition of the
// kernel depends on array contents (and it has no private arrays), so every seed of a
// launch performs the same accesses in the same rounds and only the values differ.
// tainted[v]: variable v may hold an input-dependent value (one copy per seed).
bool seed_oblivious(const Kernel& k, std::vector<bool>* tainted = nullptr);

// Block-private outputs: every global array the kernel writes is never loaded and every store
// to it has the flat index `bid.x` (casts aside).  Blocks with distinct bid.x then write
// distinct cells and read none that another block writes, so with a one-dimensional grid
// (and gdim.x <= 2^bits, the index being w-bit arithmetic, X23) no global cell is shared
// between blocks (X4 XB cannot occur): the planner drops the XB stamps and K2b for such
// launches.  The SDK reductions' `g_odata[bid.x] = sdata[0]` is the case it is for.
bool block_private_outputs(const Kernel& k);

// Thread-private stores: for each array, true when it is a one-dimensional shared array and
// every store to it has the flat index tid.x (or a variable whose every assignment is tid.x;
// casts aside).  With a one-dimensional block, two threads of a block then never store to one
// cell: no WW race on it is possible, so its stores need no ownership claim (a plain owner
// stamp), and a check needs only its reader stamps (device_rt PG_TP; the SDK reductions'
// `sdata[tid] += sdata[tid + s]`).
std::vector<bool> thread_private_stores(const Kernel& k);
// Variables holding tid.x wherever they are read: top-level aliases (thread_private_stores)
// and the hidden copies compound stores make of their index (X21).
std::vector<bool> tid_alias_vars(const Kernel& k);

}  // namespace pgf
