// ir.hpp -- in-memory form of a stencil specification (a1 output, a2 input).
//
// Mirrors the paper's minimal DSL (Listing 1, PAPER.md P:411-437 section
// II-A): declared parameters, iterators (outermost -> innermost),
// arrays and scalars, copyin/copyout (parsed and
// ignored), #pragma, #assign, one `stencil` function
// whose body is restricted C with iterator+-constant index expressions
// (P:372-378), and the call binding actuals positionally.
#pragma once

#include <array>
#include <cstdint>
#include <stdexcept>
#include <functional>
#include <map>
#include <memory>
#include <string>
#include <vector>

namespace sdag {

enum class ArgKind : int { Array3D = 0, Array1D = 1, Scalar = 2 };
enum class Role : int { In = 0, Out = 1, InOut = 2, Unused = 3 };

// Expression node.  Trees are stored in Stencil::nodes; children by index.
struct Node {
    enum Kind : int { Num, Scalar, Temp, Load3, Load1, Neg, Add, Sub, Mul, Div } kind;
    double value = 0.0;  // Num
    int ref = -1;        // Scalar: formal scalar index; Temp: temp index; Load3/Load1: formal array index
    int off[3] = {0, 0, 0};  // Load3: (dz, dy, dx); Load1: off[0] = offset along its axis
    int a = -1, b = -1;      // children
    int line = 0, col = 0;
};

struct Statement {
    bool to_array = false;  // true: writes 3D array `target` at offset 0; false: temporary `target`
    int target = -1;
    int expr = -1;          // root node
    bool declares = false;  // `double t = ...;`
    int line = 0;
};

struct Formal {
    std::string name;       // formal name inside the stencil function
    std::string actual;     // bound actual (call) -- same as name when there is no call
    ArgKind kind = ArgKind::Scalar;
    int kind_index = -1;    // position among formals of the same kind
    int axis = -1;          // 1D arrays: 0 = z, 1 = y, 2 = x (from the iterator that indexes it)
    Role role = Role::Unused;
};

struct Pragma {
    std::string stream_dim;          // "#pragma stream k"
    int block[3] = {0, 0, 0};        // block(x[,y[,z]])
    std::map<std::string, int> unroll;  // unroll j=2
    double occupancy = 0.0;          // occupancy t
};

struct Assign {
    std::vector<std::string> shmem, gmem;  // #assign shmem(...), gmem(...)
};

struct Stencil {
    std::string name;
    std::vector<std::string> iterators;  // outermost..innermost as declared
    std::map<std::string, int64_t> parameters;
    std::vector<Formal> formals;
    std::vector<std::string> temps;      // temporary scalar names
    std::vector<Node> nodes;
    std::vector<Statement> stmts;
    Pragma pragma;
    Assign assign;
    bool has_call = false;

    int n_of(ArgKind k) const {
        int n = 0;
        for (auto &f : formals) n += (f.kind == k);
        return n;
    }
    const Formal &formal(ArgKind k, int idx) const {
        for (auto &f : formals)
            if (f.kind == k && f.kind_index == idx) return f;
        static Formal none;
        return none;
    }
};

// a2 results
struct Analysis {
    int radius[3] = {0, 0, 0};            // z, y, x
    std::vector<std::array<int, 3>> arr_radius;  // per 3D formal (by kind_index)
    int n_in = 0, n_out = 0, n_inout = 0;
    double flops_per_point = 0.0;         // canonical count, reading R9
    int n_io_arrays = 0;                  // Table I "#IO arrays"
    std::vector<bool> node_varies;        // node depends on an array load
    bool homogenizable_z = false;         // P:810-830 (retiming precondition)
};

// Internal error carrying an sdag_status code (converted at the C ABI).
struct Error : std::runtime_error {
    int status;
    Error(int st, const std::string &m) : std::runtime_error(m), status(st) {}
};

// a1: parse the DSL text into a resolved Stencil (throws Error).  Specs with
// several stencil definitions or calls are programs: UNSUPPORTED here.
Stencil parse_spec(const std::string &text);

// A multi-stencil program (Fig 3c): one resolved Stencil per
// call, in call order; every stage is a full sweep over its own interior and
// sees the arrays as the previous stages left them.
struct ProgramArg {
    std::string name;  // declared name
    ArgKind kind = ArgKind::Scalar;
    int kind_index = -1;  // position among program arguments of the same kind (declaration order)
    int axis = -1;        // 1D arrays
    Role role = Role::Unused;  // program-level (filled by the planner)
};
struct ProgramIR {
    std::vector<Stencil> stages;
    std::vector<ProgramArg> args;        // declared names bound by some stage, declaration order
    std::vector<std::vector<int>> map;   // map[s][formal position] = index into args
};
ProgramIR parse_program(const std::string &text);
// a2: analyse (throws Error for UNSUPPORTED / SEMANTIC findings).
Analysis analyse(const Stencil &st);
// fission versions of a single-stage spec as DSL program text (fission.cpp):
// kind 0 maxfuse, 1 trivial-fission
std::string emit_fission(const std::string &spec, int kind);
// maxfuse of a multi-stencil program with recomputation (fission.cpp): one
// stencil; keep_intermediates = 0 writes only arrays no later stage reads
std::string fuse_program(const std::string &text, int keep_intermediates);
// Section VI-B versions of a multi-stencil program (fission.cpp): calls grouped
// in call order (sizes add up to the number of calls), each group fused with
// recomputation; recompute-fission = groups grown while the recomputation halo
// <= max(4, r); forest_partitions = every partition whose groups obey that bound
// and have <= 4 recomputed RAW intermediates (staged first, maxfuse last)
std::string fuse_groups(const std::string &text, const std::vector<int> &sizes);
std::string recompute_fission(const std::string &text, std::vector<int> *sizes_out);
std::vector<std::vector<int>> forest_partitions(const std::string &text, int max_candidates);
std::string group_report(const std::string &text, const std::vector<int> &sizes);
// canonical, name-free serialisation used to match registered DAGs
std::string canonical_form(const Stencil &st);

}  // namespace sdag
