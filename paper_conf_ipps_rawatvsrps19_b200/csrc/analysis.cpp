// analysis.cpp -- a2: footprint, per-axis radius, roles, canonical counts.
//
//  - radius: R_a = max |offset| along axis a over every read (3D and 1D)
//    (stencil order; per axis: DESIGN.md reading R2)
//  - roles: in / out / inout (read at offset 0 before its first write) and the
//    read-after-write rule of reading R1 (a later read at offset 0 sees the new
//    value; any shifted read of a written array is UNSUPPORTED)
//  - canonical flops/point (reading R9): binary + - * / count 1 each, unary
//    minus 0, and operations whose operands are all loop-invariant (scalars,
//    literals, invariant temporaries, e.g. `c = b*h2inv`, Listing 1 line 7)
//    count 0.  Pinned by Table I: jacobi 10, hypterm 358,
//    rhs4center 666.
//  - homogenizability along z (retiming precondition): after
//    distributing invariant factors over sums, every additive term reads a
//    single z-offset.
#include "ir.hpp"
#include "sdag.h"

#include <cstdio>
#include <cstdlib>
#include <functional>
#include <cstring>
#include <set>
#include <sstream>

namespace sdag {

namespace {

void terms_of(const Stencil &S, const std::vector<bool> &var, int n, std::vector<int> &out) {
    const Node &x = S.nodes[n];
    if (x.kind == Node::Add || x.kind == Node::Sub) {
        terms_of(S, var, x.a, out);
        terms_of(S, var, x.b, out);
        return;
    }
    if (x.kind == Node::Neg) {
        terms_of(S, var, x.a, out);
        return;
    }
    if (x.kind == Node::Mul || x.kind == Node::Div) {
        // distribute an invariant factor over a sum: c*(a+b) -> c*a + c*b
        bool va = var[x.a], vb = var[x.b];
        if (!va && vb && x.kind == Node::Mul) { terms_of(S, var, x.b, out); return; }
        if (va && !vb) { terms_of(S, var, x.a, out); return; }
    }
    out.push_back(n);
}

void zoffs(const Stencil &S, int n, std::set<int> &z, const std::vector<std::set<int>> &temp_z) {
    const Node &x = S.nodes[n];
    switch (x.kind) {
    case Node::Load3: z.insert(x.off[0]); break;
    case Node::Load1: break;
    case Node::Temp: z.insert(temp_z[x.ref].begin(), temp_z[x.ref].end()); break;
    default:
        if (x.a >= 0) zoffs(S, x.a, z, temp_z);
        if (x.b >= 0) zoffs(S, x.b, z, temp_z);
    }
}

}  // namespace

Analysis analyse(const Stencil &S) {
    Analysis A;
    const int n3 = S.n_of(ArgKind::Array3D);
    A.arr_radius.assign(n3, {0, 0, 0});
    A.node_varies.assign(S.nodes.size(), false);

    std::vector<bool> written(n3, false), read_before(n3, false), read_any(n3, false);
    std::vector<bool> temp_varies(S.temps.size(), false);
    std::vector<std::set<int>> temp_z(S.temps.size());
    double flops = 0.0;

    // nodes are created children-first, but temporaries depend on statement
    // order, so evaluate `varies` per statement in program order.
    std::vector<char> done(S.nodes.size(), 0);
    std::function<bool(int)> varies = [&](int n) -> bool {
        const Node &x = S.nodes[n];
        bool v = false;
        switch (x.kind) {
        case Node::Num:
        case Node::Scalar: v = false; break;
        case Node::Load3:
        case Node::Load1: v = true; break;
        case Node::Temp: v = temp_varies[x.ref]; break;
        case Node::Neg: v = varies(x.a); break;
        default: {
            bool a = varies(x.a), b = varies(x.b);
            v = a || b;
            if (v) flops += 1.0;  // binary op on a point-dependent operand
        }
        }
        A.node_varies[n] = v;
        return v;
    };

    std::function<void(int)> reads = [&](int n) {
        const Node &x = S.nodes[n];
        if (x.kind == Node::Load3) {
            int r = x.ref;
            for (int a = 0; a < 3; a++) {
                int m = std::abs(x.off[a]);
                if (m > A.radius[a]) A.radius[a] = m;
                if (m > A.arr_radius[r][a]) A.arr_radius[r][a] = m;
            }
            read_any[r] = true;
            bool zero = x.off[0] == 0 && x.off[1] == 0 && x.off[2] == 0;
            if (written[r] && !zero)
                throw Error(SDAG_ERR_UNSUPPORTED,
                            std::to_string(x.line) + ":" + std::to_string(x.col) +
                                ": shifted read of an array written earlier in the stencil (multi-stage DAG, NEXT-4)");
            if (!written[r]) read_before[r] = true;
        } else if (x.kind == Node::Load1) {
            const Formal &f = S.formal(ArgKind::Array1D, x.ref);
            int m = std::abs(x.off[0]);
            if (m > A.radius[f.axis]) A.radius[f.axis] = m;
        }
        if (x.kind >= Node::Neg) {
            reads(x.a);
            if (x.b >= 0) reads(x.b);
        }
    };

    bool homog = true;
    for (const Statement &st : S.stmts) {
        reads(st.expr);
        bool v = varies(st.expr);
        std::vector<int> terms;
        terms_of(S, A.node_varies, st.expr, terms);
        std::set<int> zall;
        for (int t : terms) {
            std::set<int> z;
            zoffs(S, t, z, temp_z);
            if (z.size() > 1) homog = false;
            zall.insert(z.begin(), z.end());
        }
        if (st.to_array) {
            written[st.target] = true;
        } else {
            temp_varies[st.target] = v;
            temp_z[st.target] = zall;
        }
    }
    // a shifted read of an array that is written LATER is also unsupported
    for (const Statement &st : S.stmts) {
        std::function<void(int)> chk = [&](int n) {
            const Node &x = S.nodes[n];
            if (x.kind == Node::Load3 && written[x.ref] && (x.off[0] || x.off[1] || x.off[2]))
                throw Error(SDAG_ERR_UNSUPPORTED, std::to_string(x.line) + ":" + std::to_string(x.col) +
                                                      ": shifted read of an array the stencil writes");
            if (x.kind == Node::Neg || x.kind >= Node::Add) {
                chk(x.a);
                if (x.b >= 0) chk(x.b);
            }
        };
        chk(st.expr);
    }
    A.flops_per_point = flops;
    A.homogenizable_z = homog;

    for (auto &f : const_cast<Stencil &>(S).formals) {
        if (f.kind != ArgKind::Array3D) continue;
        int r = f.kind_index;
        if (written[r]) f.role = read_before[r] ? Role::InOut : Role::Out;
        else f.role = read_any[r] ? Role::In : Role::Unused;
        A.n_in += f.role == Role::In;
        A.n_out += f.role == Role::Out;
        A.n_inout += f.role == Role::InOut;
    }
    A.n_io_arrays = A.n_in + A.n_out + A.n_inout;
    if (A.n_out + A.n_inout == 0) throw Error(SDAG_ERR_SEMANTIC, "the stencil writes no array");
    return A;
}

// Name-free serialisation: formal kinds in order, 1D axes, statements as
// prefix trees with literal bit patterns.  Two specs with equal canonical
// forms denote the same DAG (up to renaming), so they may share a kernel.
std::string canonical_form(const Stencil &S) {
    std::ostringstream o;
    o << "it" << S.iterators.size() << "|F";
    for (auto &f : S.formals) {
        o << (f.kind == ArgKind::Array3D ? 'G' : f.kind == ArgKind::Array1D ? 'L' : 'S');
        if (f.kind == ArgKind::Array1D) o << f.axis;
    }
    o << "|T" << S.temps.size();
    std::function<void(int)> emit = [&](int n) {
        const Node &x = S.nodes[n];
        switch (x.kind) {
        case Node::Num: {
            uint64_t b;
            std::memcpy(&b, &x.value, 8);
            char buf[32];
            std::snprintf(buf, sizeof buf, "#%016llx", (unsigned long long)b);
            o << buf;
            break;
        }
        case Node::Scalar: o << "s" << x.ref; break;
        case Node::Temp: o << "t" << x.ref; break;
        case Node::Load3: o << "g" << x.ref << "[" << x.off[0] << "," << x.off[1] << "," << x.off[2] << "]"; break;
        case Node::Load1: o << "l" << x.ref << "[" << x.off[0] << "]"; break;
        case Node::Neg: o << "(~ "; emit(x.a); o << ")"; break;
        default: {
            const char *op = x.kind == Node::Add ? "+" : x.kind == Node::Sub ? "-" : x.kind == Node::Mul ? "*" : "/";
            o << "(" << op << " ";
            emit(x.a);
            o << " ";
            emit(x.b);
            o << ")";
        }
        }
    };
    for (auto &st : S.stmts) {
        o << "|" << (st.to_array ? "G" : "t") << st.target << "=";
        emit(st.expr);
    }
    return o.str();
}

}  // namespace sdag
