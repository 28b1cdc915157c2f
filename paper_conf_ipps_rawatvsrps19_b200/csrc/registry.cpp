// registry.cpp -- the stencil DAGs that have hand-written sm_100a bodies, and
// the matcher that binds a parsed spec to one of them (a3, first step).
//
// A spec is dispatched to a registered body iff its canonical form
// (analysis.cpp: formal kinds, 1D axes, statement trees, literal bits --
// everything but names) equals that of the registered spec text in
// specs/<name>.sdag.  The shift toy accepts any single-tap translation.
#include "registry.hpp"

#include "ir.hpp"
#include "sdag.h"

#include <mutex>

namespace sdag {

namespace {

struct Embedded {
    const char *name;
    const char *text;
};

// specs_embed.inc is generated at build time from specs/*.sdag
const Embedded kSpecs[] = {
#include "specs_embed.inc"
};

std::vector<RegEntry> build() {
    std::vector<RegEntry> v;
    for (const auto &e : kSpecs) {
        RegEntry r;
        r.name = e.name;
        r.text = e.text;
        Stencil st = parse_spec(r.text);
        analyse(st);
        r.canonical = canonical_form(st);
        v.push_back(r);
    }
    return v;
}

}  // namespace

const std::vector<RegEntry> &registry() {
    static std::once_flag once;
    static std::vector<RegEntry> reg;
    std::call_once(once, [] { reg = build(); });
    return reg;
}

// Returns the matched entry (nullptr if none); extra[] receives plan-time
// kernel scalars (the shift offsets).
const RegEntry *match_dag(const Stencil &st, std::vector<double> &extra) {
    extra.clear();
    const std::string canon = canonical_form(st);
    for (const auto &r : registry()) {
        if (r.name == "shift") continue;
        if (r.canonical == canon) return &r;
    }
    // shift family: one statement G_out = G_in[dz,dy,dx], no scalars / 1D arrays
    if (st.stmts.size() == 1 && st.stmts[0].to_array && st.n_of(ArgKind::Scalar) == 0 &&
        st.n_of(ArgKind::Array1D) == 0 && st.n_of(ArgKind::Array3D) == 2 && st.iterators.size() == 3) {
        const Node &n = st.nodes[st.stmts[0].expr];
        if (n.kind == Node::Load3 && n.ref != st.stmts[0].target) {
            bool ok = true;
            for (int a = 0; a < 3; a++) ok = ok && std::abs(n.off[a]) <= 4;
            if (ok) {
                for (const auto &r : registry())
                    if (r.name == "shift") {
                        extra = {double(n.off[0]), double(n.off[1]), double(n.off[2])};
                        return &r;
                    }
            }
        }
    }
    return nullptr;
}

std::string registry_names() {
    std::string s;
    for (const auto &r : registry()) s += (s.empty() ? "" : ", ") + r.name;
    return s;
}

}  // namespace sdag
