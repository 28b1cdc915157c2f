// registry.hpp -- registered stencil DAGs (see registry.cpp).
#pragma once

#include <string>
#include <vector>

namespace sdag {

struct Stencil;

struct RegEntry {
    std::string name;       // "jacobi7", "lap25", ...
    std::string text;       // canonical DSL text (specs/<name>.sdag)
    std::string canonical;  // canonical_form() of text
};

const std::vector<RegEntry> &registry();
const RegEntry *match_dag(const Stencil &st, std::vector<double> &extra_scalars);
std::string registry_names();

}  // namespace sdag
