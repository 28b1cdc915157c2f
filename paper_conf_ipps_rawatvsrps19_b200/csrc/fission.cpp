// fission.cpp -- the paper's fission component (Section VI-B):
// from a single-stage spec, write the split versions back out as DSL text that
// sdag_program_create accepts (ARTEMIS "writes them out as DSL specification
// files"):
//   * maxfuse: the stencil itself, re-printed from the IR (every stencil
//     function with the same domain fused -- one stage here);
//   * trivial-fission: one stencil function per output array, holding the
//     statements that array needs (temporaries replicated, Fig 3b/3c), called
//     in an order that preserves every value a statement reads.
// A split is emitted only if every stage keeps the stencil's radius (each
// stage's output domain is the interior of its own radius, reading R1).
// Recompute-fission splits outputs so that each kernel's recomputation halo is
// <= max(4, r); the temporaries of this DSL are per-point scalars (reading
// R15), so a single stage has no recomputation halo and recompute-fission
// coincides with maxfuse.
//
// Statements are selected, never rewritten: each printed expression is the
// parsed tree, fully parenthesised, literals printed to round-trip exactly.
#include <algorithm>
#include <cstdio>
#include <functional>
#include <set>
#include <sstream>

#include "ir.hpp"
#include "sdag.h"

namespace sdag {

namespace {

std::string num(double v) {
    char b[40];
    std::snprintf(b, sizeof b, "%.17g", v);
    std::string s = b;
    if (s.find_first_of(".eEn") == std::string::npos) s += ".0";  // a double literal
    return s;
}

struct Printer {
    const Stencil &st;
    std::string expr(int n) const {
        const Node &x = st.nodes[n];
        switch (x.kind) {
            case Node::Num: return num(x.value);
            case Node::Scalar: return st.formal(ArgKind::Scalar, x.ref).name;
            case Node::Temp: return st.temps[x.ref];
            case Node::Load3: {
                std::string s = st.formal(ArgKind::Array3D, x.ref).name;
                for (int a = 0; a < 3; a++) s += "[" + idx(a, x.off[a]) + "]";
                return s;
            }
            case Node::Load1: {
                const Formal &f = st.formal(ArgKind::Array1D, x.ref);
                return f.name + "[" + idx(f.axis, x.off[0]) + "]";
            }
            case Node::Neg: return "(-" + expr(x.a) + ")";
            case Node::Add: return "(" + expr(x.a) + " + " + expr(x.b) + ")";
            case Node::Sub: return "(" + expr(x.a) + " - " + expr(x.b) + ")";
            case Node::Mul: return "(" + expr(x.a) + " * " + expr(x.b) + ")";
            case Node::Div: return "(" + expr(x.a) + " / " + expr(x.b) + ")";
        }
        throw Error(SDAG_ERR_INVALID_ARG, "fission: unknown node");
    }
    std::string idx(int axis, int off) const {
        const std::string &it = st.iterators[axis];
        if (off == 0) return it;
        return it + (off > 0 ? "+" : "-") + std::to_string(std::abs(off));
    }
};

// temporaries and 3D arrays (offset 0 reads) an expression reads
void reads(const Stencil &st, int n, std::set<int> &temps, std::vector<int> *arrays0) {
    const Node &x = st.nodes[n];
    if (x.kind == Node::Temp) temps.insert(x.ref);
    if (x.kind == Node::Load3 && arrays0 && x.off[0] == 0 && x.off[1] == 0 && x.off[2] == 0)
        arrays0->push_back(x.ref);
    if (x.a >= 0) reads(st, x.a, temps, arrays0);
    if (x.b >= 0) reads(st, x.b, temps, arrays0);
}

// per-axis radius of the reads of an expression (3D and 1D, reading R2)
void radius_of(const Stencil &st, int n, int r[3]) {
    const Node &x = st.nodes[n];
    if (x.kind == Node::Load3)
        for (int a = 0; a < 3; a++) r[a] = std::max(r[a], std::abs(x.off[a]));
    if (x.kind == Node::Load1) {
        const int a = st.formal(ArgKind::Array1D, x.ref).axis;
        if (a >= 0) r[a] = std::max(r[a], std::abs(x.off[0]));
    }
    if (x.a >= 0) radius_of(st, x.a, r);
    if (x.b >= 0) radius_of(st, x.b, r);
}

std::string header(const Stencil &st) {
    std::ostringstream o;
    o << "iterator";
    for (size_t a = 0; a < st.iterators.size(); a++) o << (a ? ", " : " ") << st.iterators[a];
    o << ";\n";
    // declared extents are placeholders: a plan's extents come from sdag_plan_create
    std::vector<std::string> decl;
    std::set<std::string> seen;
    for (const Formal &f : st.formals) {
        const std::string &n = f.actual.empty() ? f.name : f.actual;
        if (!seen.insert(n).second) continue;
        if (f.kind == ArgKind::Array3D)
            decl.push_back(n + "[64,64,64]");
        else if (f.kind == ArgKind::Array1D)
            decl.push_back(n + "[64]");
        else
            decl.push_back(n);
    }
    o << "double";
    for (size_t q = 0; q < decl.size(); q++) o << (q ? ", " : " ") << decl[q];
    o << ";\n";
    return o.str();
}

std::string formals_list(const Stencil &st, bool actual) {
    std::string s = "(";
    for (size_t q = 0; q < st.formals.size(); q++) {
        const Formal &f = st.formals[q];
        s += (q ? ", " : "") + ((actual && !f.actual.empty()) ? f.actual : f.name);
    }
    return s + ")";
}

std::string function(const Stencil &st, const std::string &name, const std::vector<bool> &keep) {
    Printer P{st};
    std::ostringstream o;
    o << "stencil " << name << " " << formals_list(st, false) << " {\n";
    std::set<int> declared;
    for (size_t q = 0; q < st.stmts.size(); q++) {
        if (!keep[q]) continue;
        const Statement &s = st.stmts[q];
        o << "    ";
        if (s.to_array) {
            o << st.formal(ArgKind::Array3D, s.target).name << "[" << P.idx(0, 0) << "][" << P.idx(1, 0) << "]["
              << P.idx(2, 0) << "]";
        } else {
            if (declared.insert(s.target).second) o << "double ";
            o << st.temps[s.target];
        }
        o << " = " << P.expr(s.expr) << ";\n";
    }
    o << "}\n";
    return o.str();
}

}  // namespace

std::string emit_fission(const std::string &spec, int kind) {
    const Stencil st = parse_spec(spec);
    (void)analyse(st);  // the spec must be a valid single-stage DAG
    const int ns = int(st.stmts.size());
    if (kind == 0) {  // maxfuse: the stencil re-printed
        std::vector<bool> all(ns, true);
        return header(st) + function(st, st.name, all) + st.name + " " + formals_list(st, true) + ";\n";
    }
    if (kind != 1) throw Error(SDAG_ERR_INVALID_ARG, "fission kind must be 0 (maxfuse) or 1 (trivial-fission)");

    // output arrays in order of first write
    std::vector<int> outs;
    for (const Statement &s : st.stmts)
        if (s.to_array && std::find(outs.begin(), outs.end(), s.target) == outs.end()) outs.push_back(s.target);
    const int no = int(outs.size());
    auto out_index = [&](int arr) {
        auto it = std::find(outs.begin(), outs.end(), arr);
        return it == outs.end() ? -1 : int(it - outs.begin());
    };

    // backward slice per output: keep its writes and, by liveness, the
    // temporary assignments whose values they (transitively) read
    std::vector<std::vector<bool>> keep(no, std::vector<bool>(ns, false));
    std::vector<std::set<int>> before(no);  // kernels that must run before kernel m
    for (int m = 0; m < no; m++) {
        std::set<int> live;
        for (int q = ns - 1; q >= 0; q--) {
            const Statement &s = st.stmts[q];
            const bool writes_out = s.to_array && s.target == outs[m];
            const bool defines_live = !s.to_array && live.count(s.target);
            if (!writes_out && !defines_live) continue;
            keep[m][q] = true;
            if (defines_live) live.erase(s.target);
            reads(st, s.expr, live, nullptr);
        }
        // value-order constraints: a kept statement reading another output X
        // at the point sees X's new value if X was written earlier in program
        // order (X's kernel must run first), else its old value (X's kernel
        // must run after this one)
        for (int q = 0; q < ns; q++) {
            if (!keep[m][q]) continue;
            std::set<int> tmp;
            std::vector<int> arrs;
            reads(st, st.stmts[q].expr, tmp, &arrs);
            for (int x : arrs) {
                const int j = out_index(x);
                if (j < 0 || j == m) continue;
                bool written_before = false;
                for (int r = 0; r < q; r++)
                    if (st.stmts[r].to_array && st.stmts[r].target == x) written_before = true;
                if (written_before)
                    before[m].insert(j);
                else
                    before[j].insert(m);
            }
        }
    }
    // each stage's output domain is the interior of ITS radius (reading R1):
    // a stage that reads less far than the fused stencil would write a wider
    // domain, so the split is only emitted when every stage keeps the radius
    const Analysis full = analyse(st);
    for (int m = 0; m < no; m++) {
        int r[3] = {0, 0, 0};
        for (int q = 0; q < ns; q++)
            if (keep[m][q]) radius_of(st, st.stmts[q].expr, r);
        for (int a = 0; a < 3; a++)
            if (r[a] != full.radius[a])
                throw Error(SDAG_ERR_UNSUPPORTED,
                            "trivial fission would change the output domain of '" +
                                st.formal(ArgKind::Array3D, outs[m]).name + "' (its statements read radius " +
                                std::to_string(r[a]) + " along axis " + std::to_string(a) + ", the stencil " +
                                std::to_string(full.radius[a]) + ")");
    }
    // call order: outputs' first-write order, subject to the constraints
    std::vector<int> order;
    std::vector<bool> placed(no, false);
    for (int step = 0; step < no; step++) {
        int pick = -1;
        for (int m = 0; m < no && pick < 0; m++) {
            if (placed[m]) continue;
            bool ready = true;
            for (int j : before[m]) ready = ready && placed[j];
            if (ready) pick = m;
        }
        if (pick < 0)
            throw Error(SDAG_ERR_UNSUPPORTED,
                        "trivial fission would change a value some statement reads (outputs read each other's old "
                        "and new values)");
        placed[pick] = true;
        order.push_back(pick);
    }
    std::string text = header(st), calls;
    for (int m : order) {
        const std::string name = st.name + "_" + st.formal(ArgKind::Array3D, outs[m]).name;
        text += function(st, name, keep[m]);
        calls += name + " " + formals_list(st, true) + ";\n";
    }
    return text + calls;
}

}  // namespace sdag

// ---------------------------------------------------------------------------
// maxfuse of a multi-stencil program (Section VI-B "maxfuse", P:1505-1512,
// with the recomputation the paper weighs against fusion): the
// stages are fused into ONE stencil.  A read of an array that an earlier stage
// wrote is replaced by that stage's expression for it, evaluated at the
// read's offset (temporaries inlined, shifted), so the intermediate never goes
// through memory and is recomputed once per use.  The fused stencil's radius
// is the composed one (e.g. 1 + 1 for a Laplacian of a Laplacian) and it
// writes every program output on ITS interior: there each value is computed
// by exactly the operations the staged program performs.
// ---------------------------------------------------------------------------

namespace sdag {

namespace {

struct Fuser {
    const ProgramIR &ir;
    std::vector<std::string> iters;
    int s0 = 0;  // first stage of the fused group: earlier stages' results are read from memory

    const std::string &argname(int s, int formal_pos) const { return ir.args[ir.map[s][formal_pos]].name; }
    int arg_of(int s, ArgKind k, int kind_index) const {
        const Stencil &st = ir.stages[s];
        for (size_t q = 0; q < st.formals.size(); q++)
            if (st.formals[q].kind == k && st.formals[q].kind_index == kind_index) return ir.map[s][q];
        throw Error(SDAG_ERR_INVALID_ARG, "fuse: formal not bound");
    }
    std::string idx(int axis, int off) const {
        const std::string &it = iters[axis];
        if (off == 0) return it;
        return it + (off > 0 ? "+" : "-") + std::to_string(std::abs(off));
    }
    // last statement < q of stage s writing 3D arg a (or -1)
    int last_write(int s, int a, int q) const {
        const Stencil &st = ir.stages[s];
        for (int r = q - 1; r >= 0; r--)
            if (st.stmts[r].to_array && arg_of(s, ArgKind::Array3D, st.stmts[r].target) == a) return r;
        return -1;
    }
    int last_temp(int s, int t, int q) const {
        const Stencil &st = ir.stages[s];
        for (int r = q - 1; r >= 0; r--)
            if (!st.stmts[r].to_array && st.stmts[r].target == t) return r;
        return -1;
    }
    // value of 3D arg a as stage s (before statement q) sees it, at shift d
    std::string value(int s, int q, int a, const int d[3], const std::vector<bool> &fused_writes) const {
        const int w = last_write(s, a, q);
        if (w >= 0) return "(" + expr(s, w, ir.stages[s].stmts[w].expr, d, fused_writes) + ")";
        for (int e = s - 1; e >= s0; e--) {  // the last earlier stage of the group that wrote a
            const int we = last_write(e, a, int(ir.stages[e].stmts.size()));
            if (we >= 0) return "(" + expr(e, we, ir.stages[e].stmts[we].expr, d, fused_writes) + ")";
        }
        // a program input (or an output's initial contents)
        if (fused_writes[a] && (d[0] || d[1] || d[2]))
            throw Error(SDAG_ERR_UNSUPPORTED, "fuse: array '" + ir.args[a].name +
                                                  "' is read at an offset before any stage writes it and is also "
                                                  "written by the fused stencil");
        std::string s3 = ir.args[a].name;
        for (int ax = 0; ax < 3; ax++) s3 += "[" + idx(ax, d[ax]) + "]";
        return s3;
    }
    std::string expr(int s, int q, int n, const int d[3], const std::vector<bool> &fw) const {
        const Stencil &st = ir.stages[s];
        const Node &x = st.nodes[n];
        switch (x.kind) {
            case Node::Num: return num(x.value);
            case Node::Scalar: return ir.args[arg_of(s, ArgKind::Scalar, x.ref)].name;
            case Node::Temp: {
                const int r = last_temp(s, x.ref, q);
                if (r < 0) throw Error(SDAG_ERR_SEMANTIC, "fuse: temporary read before assignment");
                return "(" + expr(s, r, st.stmts[r].expr, d, fw) + ")";
            }
            case Node::Load3: {
                const int dd[3] = {x.off[0] + d[0], x.off[1] + d[1], x.off[2] + d[2]};
                return value(s, q, arg_of(s, ArgKind::Array3D, x.ref), dd, fw);
            }
            case Node::Load1: {
                const int a = arg_of(s, ArgKind::Array1D, x.ref);
                const int ax = ir.args[a].axis;
                return ir.args[a].name + "[" + idx(ax, x.off[0] + (ax >= 0 ? d[ax] : 0)) + "]";
            }
            case Node::Neg: return "(-" + expr(s, q, x.a, d, fw) + ")";
            case Node::Add: return "(" + expr(s, q, x.a, d, fw) + " + " + expr(s, q, x.b, d, fw) + ")";
            case Node::Sub: return "(" + expr(s, q, x.a, d, fw) + " - " + expr(s, q, x.b, d, fw) + ")";
            case Node::Mul: return "(" + expr(s, q, x.a, d, fw) + " * " + expr(s, q, x.b, d, fw) + ")";
            case Node::Div: return "(" + expr(s, q, x.a, d, fw) + " / " + expr(s, q, x.b, d, fw) + ")";
        }
        throw Error(SDAG_ERR_INVALID_ARG, "fuse: unknown node");
    }
};

}  // namespace

std::string fuse_program(const std::string &text, int keep_intermediates) {
    const ProgramIR ir = parse_program(text);
    if (ir.stages.empty()) throw Error(SDAG_ERR_INVALID_ARG, "fuse: empty program");
    for (const Stencil &st : ir.stages) {
        (void)analyse(st);
        if (st.iterators != ir.stages[0].iterators || st.iterators.size() != 3)
            throw Error(SDAG_ERR_UNSUPPORTED, "fuse: stages must share three iterators");
    }
    Fuser F{ir, ir.stages[0].iterators, 0};
    const int na = int(ir.args.size());
    // arrays some stage writes, in order of their last write; read later?
    std::vector<bool> written(na, false), read_later(na, false);
    std::vector<std::pair<int, int>> last;  // (stage, arg) of each written arg's final write
    for (size_t s = 0; s < ir.stages.size(); s++) {
        const Stencil &st = ir.stages[s];
        for (const Statement &w : st.stmts)
            if (w.to_array) written[F.arg_of(int(s), ArgKind::Array3D, w.target)] = true;
    }
    for (size_t s = 0; s < ir.stages.size(); s++) {
        const Stencil &st = ir.stages[s];
        for (const Node &n : st.nodes)
            if (n.kind == Node::Load3) {
                const int a = F.arg_of(int(s), ArgKind::Array3D, n.ref);
                for (size_t e = 0; e < s; e++)
                    if (F.last_write(int(e), a, int(ir.stages[e].stmts.size())) >= 0) read_later[a] = true;
            }
    }
    std::vector<bool> fw(na, false);  // arrays the fused stencil writes
    for (int a = 0; a < na; a++) fw[a] = written[a] && (keep_intermediates || !read_later[a]);
    std::ostringstream o;
    o << "iterator " << F.iters[0] << ", " << F.iters[1] << ", " << F.iters[2] << ";\ndouble";
    bool first = true;
    for (const ProgramArg &a : ir.args) {
        o << (first ? " " : ", ") << a.name;
        if (a.kind == ArgKind::Array3D) o << "[64,64,64]";
        if (a.kind == ArgKind::Array1D) o << "[64]";
        first = false;
    }
    o << ";\nstencil fused (";
    for (int a = 0; a < na; a++) o << (a ? ", " : "") << ir.args[a].name;
    o << ") {\n";
    const int zero[3] = {0, 0, 0};
    int nout = 0;
    for (int a = 0; a < na; a++) {
        if (!fw[a]) continue;
        // the final value: the last stage writing a, after all its statements
        for (int s = int(ir.stages.size()) - 1; s >= 0; s--) {
            const int w = F.last_write(s, a, int(ir.stages[s].stmts.size()));
            if (w < 0) continue;
            o << "    " << ir.args[a].name << "[" << F.iters[0] << "][" << F.iters[1] << "][" << F.iters[2]
              << "] = " << F.expr(s, w, ir.stages[s].stmts[w].expr, zero, fw) << ";\n";
            nout++;
            break;
        }
    }
    if (!nout) throw Error(SDAG_ERR_SEMANTIC, "fuse: the program writes no array");
    o << "}\nfused (";
    for (int a = 0; a < na; a++) o << (a ? ", " : "") << ir.args[a].name;
    o << ");\n";
    return o.str();
}


// ---------------------------------------------------------------------------
// Recompute-fission and the fusion forest (Section VI-B).
//
// A version of a multi-stencil program is a partition of its calls (in call
// order) into contiguous groups -- the trees of the paper's forest; each group
// becomes one stencil, fused with recomputation as fuse_program does (a read
// of an array written earlier IN THE GROUP is replaced by the writer's
// expression at the read's offset; arrays written by earlier groups are read
// from memory).  A group writes the arrays a later group reads, and every
// array no later stage reads (the program's results); intermediates consumed
// only inside the group never go through memory.
//
// Per group (group_info): r = the largest stencil order (radius, reading R2)
// of its calls; halo = the recomputation halo: how far beyond an output point
// an intermediate of the group must be recomputed (a chain lap(lap(A)) of
// order-1 calls: 1); raw = the number of intermediates the group reads at a
// nonzero offset (the "RAW dependences that increase recomputation volume").
// recompute-fission: grow each group in call order while its
// halo stays <= max(4, r).  The forest search enumerates every
// partition whose groups have halo <= max(4, r) and raw <= 4 -- maxfuse, the
// staged program and everything between -- for the measured pick.
// ---------------------------------------------------------------------------

namespace {

struct Grp {
    int halo = 0, r = 0, raw = 0;
    bool ok = true;
};

Grp group_info(const ProgramIR &ir, int s0, int s1) {
    Fuser F{ir, ir.stages[0].iterators, s0};
    const int na = int(ir.args.size());
    Grp g;
    std::vector<int> need(na, -1);  // halo at which a group-internal array's values are needed
    std::vector<bool> written(na, false);
    for (int s = s0; s < s1; s++) {
        const Stencil &st = ir.stages[s];
        const Analysis an = analyse(st);
        g.r = std::max({g.r, an.radius[0], an.radius[1], an.radius[2]});
    }
    // arrays read by a later stage of the group (intermediates) and their writers
    std::vector<int> writer(na, -1);
    for (int s = s0; s < s1; s++)
        for (const Statement &w : ir.stages[s].stmts)
            if (w.to_array) writer[F.arg_of(s, ArgKind::Array3D, w.target)] = s;
    // reverse pass: a stage runs wherever one of its outputs is needed
    std::vector<int> stage_need(s1, 0);
    for (int s = s1 - 1; s >= s0; s--) {
        const Stencil &st = ir.stages[s];
        int ns = 0;
        for (const Statement &w : st.stmts)
            if (w.to_array) {
                const int a = F.arg_of(s, ArgKind::Array3D, w.target);
                if (need[a] > ns) ns = need[a];
            }
        stage_need[s] = ns;
        std::set<int> raw_here;
        for (const Node &n : st.nodes) {
            if (n.kind != Node::Load3) continue;
            const int a = F.arg_of(s, ArgKind::Array3D, n.ref);
            int e = -1;  // the group's last writer of a before stage s
            for (int q = s - 1; q >= s0; q--)
                if (F.last_write(q, a, int(ir.stages[q].stmts.size())) >= 0) {
                    e = q;
                    break;
                }
            if (e < 0) continue;
            const int d = std::max({std::abs(n.off[0]), std::abs(n.off[1]), std::abs(n.off[2])});
            need[a] = std::max(need[a], ns + d);
            if (d > 0) raw_here.insert(a);
        }
        g.raw += int(raw_here.size());
    }
    for (int a = 0; a < na; a++)
        if (need[a] > g.halo) g.halo = need[a];
    return g;
}

bool group_fusable(const ProgramIR &ir, int s0, int s1, Grp *out) {
    Grp g = group_info(ir, s0, s1);
    if (out) *out = g;
    if (s1 - s0 == 1) return true;
    return g.halo <= std::max(4, g.r) && g.raw <= 4;
}

// the group's stencil text (function `name`, formals = every program argument)
std::string group_function(const ProgramIR &ir, int s0, int s1, const std::string &name) {
    Fuser F{ir, ir.stages[0].iterators, s0};
    const int na = int(ir.args.size());
    std::vector<bool> written(na, false), read_after(na, false);
    for (int s = s0; s < s1; s++)
        for (const Statement &w : ir.stages[s].stmts)
            if (w.to_array) written[F.arg_of(s, ArgKind::Array3D, w.target)] = true;
    for (size_t s = s1; s < ir.stages.size(); s++)
        for (const Node &n : ir.stages[s].nodes)
            if (n.kind == Node::Load3) read_after[F.arg_of(int(s), ArgKind::Array3D, n.ref)] = true;
    // inside the group, is a read by a later stage of the group -> intermediate
    std::vector<bool> read_in_group(na, false);
    for (int s = s0; s < s1; s++)
        for (const Node &n : ir.stages[s].nodes)
            if (n.kind == Node::Load3) {
                const int a = F.arg_of(s, ArgKind::Array3D, n.ref);
                for (int q = s0; q < s; q++)
                    if (F.last_write(q, a, int(ir.stages[q].stmts.size())) >= 0) read_in_group[a] = true;
            }
    std::vector<bool> fw(na, false);
    for (int a = 0; a < na; a++) fw[a] = written[a] && (read_after[a] || !read_in_group[a]);
    std::ostringstream o;
    o << "stencil " << name << " (";
    for (int a = 0; a < na; a++) o << (a ? ", " : "") << ir.args[a].name;
    o << ") {\n";
    const int zero[3] = {0, 0, 0};
    for (int a = 0; a < na; a++) {
        if (!fw[a]) continue;
        for (int s = s1 - 1; s >= s0; s--) {
            const int w = F.last_write(s, a, int(ir.stages[s].stmts.size()));
            if (w < 0) continue;
            o << "    " << ir.args[a].name << "[" << F.iters[0] << "][" << F.iters[1] << "][" << F.iters[2]
              << "] = " << F.expr(s, w, ir.stages[s].stmts[w].expr, zero, fw) << ";\n";
            break;
        }
    }
    o << "}\n";
    return o.str();
}

std::string program_of_groups(const ProgramIR &ir, const std::vector<int> &sizes) {
    const auto &it = ir.stages[0].iterators;
    std::ostringstream o;
    o << "iterator " << it[0] << ", " << it[1] << ", " << it[2] << ";\ndouble";
    bool first = true;
    for (const ProgramArg &a : ir.args) {
        o << (first ? " " : ", ") << a.name;
        if (a.kind == ArgKind::Array3D) o << "[64,64,64]";
        if (a.kind == ArgKind::Array1D) o << "[64]";
        first = false;
    }
    o << ";\n";
    int s0 = 0, gi = 0;
    std::ostringstream calls;
    for (int n : sizes) {
        const std::string name = "g" + std::to_string(gi++);
        if (n == 1) {  // an unfused call: the stage itself, statements and temporaries as written
            const Stencil &st = ir.stages[s0];
            o << function(st, name, std::vector<bool>(st.stmts.size(), true));
            calls << name << " " << formals_list(st, true) << ";\n";
        } else {
            o << group_function(ir, s0, s0 + n, name);
            calls << name << " (";
            for (size_t a = 0; a < ir.args.size(); a++) calls << (a ? ", " : "") << ir.args[a].name;
            calls << ");\n";
        }
        s0 += n;
    }
    o << calls.str();
    return o.str();
}

ProgramIR checked_program(const std::string &text) {
    ProgramIR ir = parse_program(text);
    if (ir.stages.empty()) throw Error(SDAG_ERR_INVALID_ARG, "empty program");
    for (const Stencil &st : ir.stages) {
        (void)analyse(st);
        if (st.iterators != ir.stages[0].iterators || st.iterators.size() != 3)
            throw Error(SDAG_ERR_UNSUPPORTED, "stages must share three iterators");
    }
    return ir;
}

}  // namespace

std::string fuse_groups(const std::string &text, const std::vector<int> &sizes) {
    const ProgramIR ir = checked_program(text);
    int n = 0;
    for (int x : sizes) {
        if (x < 1) throw Error(SDAG_ERR_INVALID_ARG, "group sizes must be >= 1");
        n += x;
    }
    if (n != int(ir.stages.size()))
        throw Error(SDAG_ERR_INVALID_ARG, "group sizes must add up to the number of calls (" +
                                              std::to_string(ir.stages.size()) + ")");
    const std::string out = program_of_groups(ir, sizes);
    (void)checked_program(out);  // every group must be a valid stencil (e.g. no shifted self-reads)
    return out;
}

std::string recompute_fission(const std::string &text, std::vector<int> *sizes_out) {
    const ProgramIR ir = checked_program(text);
    const int ns = int(ir.stages.size());
    std::vector<int> sizes;
    int s0 = 0;
    while (s0 < ns) {
        int s1 = s0 + 1;
        while (s1 < ns && group_fusable(ir, s0, s1 + 1, nullptr)) {
            // the grown group must still be a valid fused stencil
            try {
                std::vector<int> trial(sizes);
                trial.push_back(s1 + 1 - s0);
                int rest = ns - (s1 + 1);
                for (int q = 0; q < rest; q++) trial.push_back(1);
                (void)checked_program(program_of_groups(ir, trial));
            } catch (const Error &) {
                break;
            }
            s1++;
        }
        sizes.push_back(s1 - s0);
        s0 = s1;
    }
    if (sizes_out) *sizes_out = sizes;
    return program_of_groups(ir, sizes);
}

std::vector<std::vector<int>> forest_partitions(const std::string &text, int max_candidates) {
    const ProgramIR ir = checked_program(text);
    const int ns = int(ir.stages.size());
    if (ns > 16) throw Error(SDAG_ERR_UNSUPPORTED, "forest search: more than 16 calls");
    std::vector<std::vector<int>> out;
    // every composition of ns into contiguous groups, staged first, maxfuse last
    std::vector<int> cur;
    std::function<void(int)> rec = [&](int s0) {
        if (int(out.size()) >= max_candidates) return;
        if (s0 == ns) {
            try {
                (void)checked_program(program_of_groups(ir, cur));
                out.push_back(cur);
            } catch (const Error &) {
            }
            return;
        }
        for (int n = 1; s0 + n <= ns; n++) {
            if (!group_fusable(ir, s0, s0 + n, nullptr)) break;
            cur.push_back(n);
            rec(s0 + n);
            cur.pop_back();
        }
    };
    rec(0);
    return out;
}

std::string group_report(const std::string &text, const std::vector<int> &sizes) {
    const ProgramIR ir = checked_program(text);
    std::ostringstream o;
    int s0 = 0;
    for (int n : sizes) {
        Grp g = group_info(ir, s0, s0 + n);
        o << "[" << s0 << "," << s0 + n << ") r=" << g.r << " halo=" << g.halo << " raw=" << g.raw << "\n";
        s0 += n;
    }
    return o.str();
}

}  // namespace sdag
