// spec.cpp -- a1: lexer and recursive-descent parser for the stencil DSL.
//
// Grammar (Listing 1, section II-A, plus the ARTEMIS
// extensions of section II-B and 1D arrays of P:451-455):
//   spec   := { item }
//   item   := 'parameter' ID '=' INT {',' ID '=' INT} ';'
//           | 'iterator' ID {',' ID} ';'      outermost..innermost
//           | 'double' decl {',' decl} ';'    decl := ID ['[' dims ']']
//           | ('copyin'|'copyout') ID {',' ID} ';'  (parsed, ignored)
//           | '#pragma' ... EOL
//           | 'stencil' ID '(' ids ')' '{' { stmt } '}'
//           | ID '(' ids ')' ';'              call, positional binding
// A spec with one stencil and at most one call is a plan (parse_spec); several
// stencil definitions and calls in sequence are a program (Fig 3c, P:1349-1368;
// parse_program), each call one stage.
//   stmt   := '#assign' ... EOL
//           | ['double'] lhs ('='|'+='|'-='|'*='|'/=') expr ';'
//   expr   := C precedence over + - * / unary-, parentheses, literals,
//             scalars, temporaries, X[k+c][j+c][i+c], s[i+c]
#include "ir.hpp"
#include "sdag.h"

#include <cctype>
#include <cstdlib>
#include <memory>
#include <set>
#include <sstream>

namespace sdag {
namespace {

struct Tok {
    enum K { Id, Num, Punct, Pragma, AssignLine, End } k;
    std::string s;
    int line, col;
};

std::string where(int line, int col) {
    std::ostringstream o;
    o << line << ":" << col;
    return o.str();
}

[[noreturn]] void fail(int st, int line, int col, const std::string &msg) {
    throw Error(st, where(line, col) + ": " + msg);
}

std::vector<Tok> lex(const std::string &t) {
    std::vector<Tok> out;
    size_t i = 0;
    int line = 1, col = 1;
    auto adv = [&](size_t n) {
        for (size_t q = 0; q < n && i < t.size(); q++, i++) {
            if (t[i] == '\n') { line++; col = 1; } else col++;
        }
    };
    while (i < t.size()) {
        char c = t[i];
        if (c == '\n' || c == ' ' || c == '\t' || c == '\r') { adv(1); continue; }
        if (c == '/' && i + 1 < t.size() && t[i + 1] == '/') {
            while (i < t.size() && t[i] != '\n') adv(1);
            continue;
        }
        if (c == '/' && i + 1 < t.size() && t[i + 1] == '*') {
            int l0 = line, c0 = col;
            adv(2);
            while (i + 1 < t.size() && !(t[i] == '*' && t[i + 1] == '/')) adv(1);
            if (i + 1 >= t.size()) fail(SDAG_ERR_PARSE, l0, c0, "unterminated comment");
            adv(2);
            continue;
        }
        int l0 = line, c0 = col;
        if (c == '#') {
            size_t e = t.find('\n', i);
            if (e == std::string::npos) e = t.size();
            std::string body = t.substr(i, e - i);
            Tok k{Tok::Pragma, body, l0, c0};
            if (body.rfind("#assign", 0) == 0) k.k = Tok::AssignLine;
            else if (body.rfind("#pragma", 0) != 0) fail(SDAG_ERR_PARSE, l0, c0, "unknown directive '" + body + "'");
            out.push_back(k);
            adv(e - i);
            continue;
        }
        if (std::isalpha((unsigned char)c) || c == '_') {
            size_t j = i;
            while (j < t.size() && (std::isalnum((unsigned char)t[j]) || t[j] == '_')) j++;
            out.push_back({Tok::Id, t.substr(i, j - i), l0, c0});
            adv(j - i);
            continue;
        }
        if (std::isdigit((unsigned char)c) || (c == '.' && i + 1 < t.size() && std::isdigit((unsigned char)t[i + 1]))) {
            size_t j = i;
            while (j < t.size() && std::isdigit((unsigned char)t[j])) j++;
            if (j < t.size() && t[j] == '.') {
                j++;
                while (j < t.size() && std::isdigit((unsigned char)t[j])) j++;
            }
            if (j < t.size() && (t[j] == 'e' || t[j] == 'E')) {
                size_t q = j + 1;
                if (q < t.size() && (t[q] == '+' || t[q] == '-')) q++;
                if (q < t.size() && std::isdigit((unsigned char)t[q])) {
                    j = q;
                    while (j < t.size() && std::isdigit((unsigned char)t[j])) j++;
                }
            }
            out.push_back({Tok::Num, t.substr(i, j - i), l0, c0});
            adv(j - i);
            continue;
        }
        static const char *two[] = {"+=", "-=", "*=", "/="};
        bool got = false;
        for (auto op : two)
            if (t.compare(i, 2, op) == 0) {
                out.push_back({Tok::Punct, op, l0, c0});
                adv(2);
                got = true;
                break;
            }
        if (got) continue;
        if (std::string("()[]{},;=+-*/").find(c) != std::string::npos) {
            out.push_back({Tok::Punct, std::string(1, c), l0, c0});
            adv(1);
            continue;
        }
        fail(SDAG_ERR_PARSE, l0, c0, std::string("unexpected character '") + c + "'");
    }
    out.push_back({Tok::End, "", line, col});
    return out;
}

// ---- raw (unresolved) syntax --------------------------------------------------

struct RawIdx {
    std::string iter;  // empty: integer literal index
    int off = 0;
    int line = 0, col = 0;
};

struct Raw {
    enum K { Num, Name, Neg, Bin } k;
    std::string s;  // Num text / Name / Bin op
    std::vector<RawIdx> idx;
    bool indexed = false;
    std::unique_ptr<Raw> a, b;
    int line = 0, col = 0;
};

struct RawStmt {
    bool declares = false;
    std::string lhs;
    std::vector<RawIdx> lidx;
    bool lindexed = false;
    std::string op;
    std::unique_ptr<Raw> rhs;
    int line = 0, col = 0;
};

struct Decl {
    std::vector<std::string> dims;  // empty: scalar
    int line = 0, col = 0;
};

struct Parser {
    std::vector<Tok> tk;
    size_t p = 0;

    std::map<std::string, int64_t> params;
    std::vector<std::string> iters;
    std::map<std::string, Decl> decls;
    std::vector<std::string> decl_order;

    struct Def {  // one `stencil` definition
        std::string name;
        std::vector<std::string> formals;
        std::vector<RawStmt> body;
        Pragma pragma;
        Assign assign;
        int line = 0, col = 0;
    };
    struct Call {  // one call, actuals bound positionally
        std::string name;
        std::vector<std::string> actuals;
        int line = 0, col = 0;
    };
    std::vector<Def> defs;
    std::vector<Call> calls;
    Pragma pending_pragma;
    bool have_pending_pragma = false;

    const Def *def_of(const std::string &n) const {
        for (auto &d : defs)
            if (d.name == n) return &d;
        return nullptr;
    }

    const Tok &cur() const { return tk[p]; }
    bool is(const char *s) const { return (cur().k == Tok::Punct || cur().k == Tok::Id) && cur().s == s; }
    [[noreturn]] void err(const std::string &m) const { fail(SDAG_ERR_PARSE, cur().line, cur().col, m); }
    void expect(const char *s) {
        if (!is(s)) err(std::string("expected '") + s + "', found '" + cur().s + "'");
        p++;
    }
    std::string ident() {
        if (cur().k != Tok::Id) err("expected identifier, found '" + cur().s + "'");
        return tk[p++].s;
    }
    int64_t integer() {
        bool neg = false;
        if (is("-")) { neg = true; p++; }
        if (cur().k != Tok::Num || cur().s.find_first_of(".eE") != std::string::npos)
            err("expected integer, found '" + cur().s + "'");
        int64_t v = std::strtoll(tk[p++].s.c_str(), nullptr, 10);
        return neg ? -v : v;
    }

    void parse() {
        while (cur().k != Tok::End) item();
    }

    void declare(const std::string &n, Decl d) {
        if (decls.count(n) || params.count(n))
            fail(SDAG_ERR_SEMANTIC, d.line, d.col, "'" + n + "' declared twice");
        decls[n] = d;
        decl_order.push_back(n);
    }

    void item() {
        const Tok &t = cur();
        if (t.k == Tok::Pragma) {
            pending_pragma = parse_pragma(t);
            have_pending_pragma = true;
            p++;
            return;
        }
        if (t.k == Tok::AssignLine) fail(SDAG_ERR_PARSE, t.line, t.col, "#assign outside a stencil body");
        if (t.k != Tok::Id) err("expected a declaration, stencil or call, found '" + t.s + "'");
        if (t.s == "parameter") {
            p++;
            do {
                int l = cur().line, c = cur().col;
                std::string n = ident();
                expect("=");
                int64_t v = integer();
                if (params.count(n) || decls.count(n)) fail(SDAG_ERR_SEMANTIC, l, c, "'" + n + "' declared twice");
                params[n] = v;
            } while (is(",") && (p++, true));
            expect(";");
        } else if (t.s == "iterator") {
            p++;
            if (!iters.empty()) err("iterators declared twice");
            do iters.push_back(ident());
            while (is(",") && (p++, true));
            expect(";");
            if (iters.size() > 3) fail(SDAG_ERR_UNSUPPORTED, t.line, t.col, "more than 3 iterators");
        } else if (t.s == "double" || t.s == "float" || t.s == "int") {
            if (t.s != "double")
                fail(SDAG_ERR_UNSUPPORTED, t.line, t.col, "only 'double' (FP64) data is supported");
            p++;
            do {
                Decl d;
                d.line = cur().line;
                d.col = cur().col;
                std::string n = ident();
                if (is("[")) {
                    // double in[L,M,N]  or  double in[L][M][N]
                    while (is("[")) {
                        p++;
                        do {
                            if (cur().k == Tok::Id || cur().k == Tok::Num) d.dims.push_back(tk[p++].s);
                            else err("expected dimension");
                        } while (is(",") && (p++, true));
                        expect("]");
                    }
                }
                declare(n, d);
            } while (is(",") && (p++, true));
            expect(";");
        } else if (t.s == "copyin" || t.s == "copyout") {
            p++;  // host<->device lists: the caller owns device memory
            do ident();
            while (is(",") && (p++, true));
            expect(";");
        } else if (t.s == "stencil") {
            p++;
            Def d;
            d.line = cur().line;
            d.col = cur().col;
            d.name = ident();
            if (def_of(d.name)) fail(SDAG_ERR_SEMANTIC, d.line, d.col, "stencil '" + d.name + "' defined twice");
            if (have_pending_pragma) {
                d.pragma = pending_pragma;
                have_pending_pragma = false;
            }
            expect("(");
            if (!is(")")) {
                do d.formals.push_back(ident());
                while (is(",") && (p++, true));
            }
            expect(")");
            expect("{");
            defs.push_back(std::move(d));
            while (!is("}")) {
                if (cur().k == Tok::End) err("unterminated stencil body");
                stmt();
            }
            expect("}");
        } else {
            // call: name(actuals);
            Call cl;
            cl.line = t.line;
            cl.col = t.col;
            cl.name = ident();
            if (!is("(")) fail(SDAG_ERR_PARSE, cl.line, cl.col, "unknown statement '" + cl.name + "'");
            p++;
            if (!def_of(cl.name))
                fail(SDAG_ERR_SEMANTIC, cl.line, cl.col, "call of undefined stencil '" + cl.name + "'");
            if (!is(")")) {
                do cl.actuals.push_back(ident());
                while (is(",") && (p++, true));
            }
            expect(")");
            expect(";");
            calls.push_back(std::move(cl));
        }
    }

    Pragma parse_pragma(const Tok &t) {
        // #pragma stream k block (32,16) unroll j=2 [occupancy 0.5]
        Pragma pr;
        std::vector<Tok> sub = lex(t.s.substr(7));
        for (auto &s : sub) { s.line = t.line; s.col = t.col; }
        size_t q = 0;
        auto need = [&](bool ok, const char *m) {
            if (!ok) fail(SDAG_ERR_PARSE, t.line, t.col, std::string("#pragma: ") + m);
        };
        while (sub[q].k != Tok::End) {
            need(sub[q].k == Tok::Id, "expected clause");
            std::string cl = sub[q++].s;
            if (cl == "stream") {
                need(sub[q].k == Tok::Id, "stream needs an iterator");
                pr.stream_dim = sub[q++].s;
            } else if (cl == "block") {
                need(sub[q].s == "(", "block(...)");
                q++;
                int n = 0;
                while (sub[q].k == Tok::Num && n < 3) {
                    pr.block[n++] = std::atoi(sub[q++].s.c_str());
                    if (sub[q].s == ",") q++;
                }
                need(sub[q].s == ")", "block(...)");
                q++;
            } else if (cl == "unroll") {
                while (sub[q].k == Tok::Id && sub[q + 1].s == "=") {
                    std::string it = sub[q].s;
                    need(sub[q + 2].k == Tok::Num, "unroll it=N");
                    pr.unroll[it] = std::atoi(sub[q + 2].s.c_str());
                    q += 3;
                    if (sub[q].s == ",") q++;
                }
            } else if (cl == "occupancy") {
                need(sub[q].k == Tok::Num, "occupancy t");
                pr.occupancy = std::strtod(sub[q++].s.c_str(), nullptr);
                need(pr.occupancy > 0 && pr.occupancy <= 1, "occupancy must be in (0,1]");
            } else {
                fail(SDAG_ERR_PARSE, t.line, t.col, "#pragma: unknown clause '" + cl + "'");
            }
        }
        return pr;
    }

    void parse_assign(const Tok &t) {
        std::vector<Tok> sub = lex(t.s.substr(7));
        size_t q = 0;
        while (sub[q].k != Tok::End) {
            if (sub[q].k != Tok::Id) fail(SDAG_ERR_PARSE, t.line, t.col, "#assign: expected shmem/gmem");
            std::string kind = sub[q++].s;
            if (kind != "shmem" && kind != "gmem") fail(SDAG_ERR_PARSE, t.line, t.col, "#assign: unknown " + kind);
            if (sub[q].s != "(") fail(SDAG_ERR_PARSE, t.line, t.col, "#assign: expected (");
            q++;
            while (sub[q].k == Tok::Id) {
                (kind == "shmem" ? defs.back().assign.shmem : defs.back().assign.gmem).push_back(sub[q++].s);
                if (sub[q].s == ",") q++;
            }
            if (sub[q].s != ")") fail(SDAG_ERR_PARSE, t.line, t.col, "#assign: expected )");
            q++;
            if (sub[q].s == ",") q++;
        }
    }

    std::vector<RawIdx> indices() {
        std::vector<RawIdx> v;
        while (is("[")) {
            p++;
            RawIdx r;
            r.line = cur().line;
            r.col = cur().col;
            // iterator [+|- INT]  |  INT [+ iterator]  |  INT
            if (cur().k == Tok::Id) {
                r.iter = ident();
                if (is("+") || is("-")) {
                    bool neg = is("-");
                    p++;
                    int64_t c = integer();
                    r.off = int(neg ? -c : c);
                }
            } else {
                int64_t c = integer();
                if (is("+")) {
                    p++;
                    r.iter = ident();
                }
                r.off = int(c);
            }
            expect("]");
            v.push_back(r);
        }
        return v;
    }

    void stmt() {
        const Tok &t = cur();
        if (t.k == Tok::AssignLine) {
            parse_assign(t);
            p++;
            return;
        }
        if (t.k == Tok::Pragma) fail(SDAG_ERR_PARSE, t.line, t.col, "#pragma inside a stencil body");
        RawStmt s;
        s.line = t.line;
        s.col = t.col;
        if (is("double")) {
            s.declares = true;
            p++;
        }
        s.lhs = ident();
        if (is("[")) {
            s.lindexed = true;
            s.lidx = indices();
        }
        if (is("=") || is("+=") || is("-=") || is("*=") || is("/=")) s.op = tk[p++].s;
        else err("expected assignment");
        if (s.declares && s.op != "=") err("declaration needs '='");
        s.rhs = expr();
        expect(";");
        defs.back().body.push_back(std::move(s));
    }

    std::unique_ptr<Raw> expr() {
        auto l = term();
        while (is("+") || is("-")) {
            auto n = std::make_unique<Raw>();
            n->k = Raw::Bin;
            n->line = cur().line;
            n->col = cur().col;
            n->s = tk[p++].s;
            n->a = std::move(l);
            n->b = term();
            l = std::move(n);
        }
        return l;
    }
    std::unique_ptr<Raw> term() {
        auto l = unary();
        while (is("*") || is("/")) {
            auto n = std::make_unique<Raw>();
            n->k = Raw::Bin;
            n->line = cur().line;
            n->col = cur().col;
            n->s = tk[p++].s;
            n->a = std::move(l);
            n->b = unary();
            l = std::move(n);
        }
        return l;
    }
    std::unique_ptr<Raw> unary() {
        if (is("-")) {
            auto n = std::make_unique<Raw>();
            n->k = Raw::Neg;
            n->line = cur().line;
            n->col = cur().col;
            p++;
            n->a = unary();
            return n;
        }
        if (is("+")) {
            p++;
            return unary();
        }
        return primary();
    }
    std::unique_ptr<Raw> primary() {
        auto n = std::make_unique<Raw>();
        n->line = cur().line;
        n->col = cur().col;
        if (is("(")) {
            p++;
            auto e = expr();
            expect(")");
            return e;
        }
        if (cur().k == Tok::Num) {
            n->k = Raw::Num;
            n->s = tk[p++].s;
            return n;
        }
        if (cur().k == Tok::Id) {
            n->k = Raw::Name;
            n->s = ident();
            if (is("[")) {
                n->indexed = true;
                n->idx = indices();
            }
            return n;
        }
        err("expected expression, found '" + cur().s + "'");
    }
};

// ---- resolution -------------------------------------------------------------

struct Resolver {
    const Parser &P;
    const Parser::Def &D;
    const Parser::Call *C;  // null: the definition evaluated on its own formals
    Stencil &S;
    std::map<std::string, int> formal_of;  // formal name -> index in S.formals
    std::map<std::string, int> temp_of;
    std::set<std::string> temp_assigned;
    int n_iter = 0;

    Resolver(const Parser &p, const Parser::Def &d, const Parser::Call *c, Stencil &s) : P(p), D(d), C(c), S(s) {}

    int iter_pos(const std::string &it) const {
        for (int q = 0; q < n_iter; q++)
            if (P.iters[q] == it) return q;
        return -1;
    }
    // grid axis (0=z,1=y,2=x) of iterator position q among n_iter iterators
    int axis_of_pos(int q) const { return 3 - n_iter + q; }

    int add(Node n) {
        S.nodes.push_back(n);
        return int(S.nodes.size()) - 1;
    }

    int resolve(const Raw &r) {
        Node n;
        n.line = r.line;
        n.col = r.col;
        switch (r.k) {
        case Raw::Num: {
            n.kind = Node::Num;
            char *end = nullptr;
            n.value = std::strtod(r.s.c_str(), &end);  // correctly rounded (reading R4)
            return add(n);
        }
        case Raw::Neg:
            n.kind = Node::Neg;
            n.a = resolve(*r.a);
            return add(n);
        case Raw::Bin: {
            n.kind = r.s == "+" ? Node::Add : r.s == "-" ? Node::Sub : r.s == "*" ? Node::Mul : Node::Div;
            n.a = resolve(*r.a);
            n.b = resolve(*r.b);
            return add(n);
        }
        case Raw::Name:
            break;
        }
        // names
        if (!r.indexed) {
            auto t = temp_of.find(r.s);
            if (t != temp_of.end()) {
                if (!temp_assigned.count(r.s))
                    fail(SDAG_ERR_SEMANTIC, r.line, r.col, "temporary '" + r.s + "' read before assignment");
                n.kind = Node::Temp;
                n.ref = t->second;
                return add(n);
            }
            auto f = formal_of.find(r.s);
            if (f == formal_of.end()) {
                if (iter_pos(r.s) >= 0)
                    fail(SDAG_ERR_UNSUPPORTED, r.line, r.col, "iterator '" + r.s + "' used as a value");
                fail(SDAG_ERR_SEMANTIC, r.line, r.col, "undeclared name '" + r.s + "'");
            }
            const Formal &fo = S.formals[f->second];
            if (fo.kind != ArgKind::Scalar)
                fail(SDAG_ERR_SEMANTIC, r.line, r.col, "array '" + r.s + "' used without an index");
            n.kind = Node::Scalar;
            n.ref = fo.kind_index;
            return add(n);
        }
        auto f = formal_of.find(r.s);
        if (f == formal_of.end()) fail(SDAG_ERR_SEMANTIC, r.line, r.col, "undeclared array '" + r.s + "'");
        Formal &fo = S.formals[f->second];
        if (fo.kind == ArgKind::Scalar)
            fail(SDAG_ERR_SEMANTIC, r.line, r.col, "scalar '" + r.s + "' indexed");
        if (fo.kind == ArgKind::Array3D) {
            if ((int)r.idx.size() != n_iter)
                fail(SDAG_ERR_SEMANTIC, r.line, r.col,
                     "grid array '" + r.s + "' needs " + std::to_string(n_iter) + " indices");
            n.kind = Node::Load3;
            n.ref = fo.kind_index;
            for (int q = 0; q < n_iter; q++) {
                const RawIdx &ix = r.idx[q];
                int pos = iter_pos(ix.iter);
                if (ix.iter.empty() || pos < 0)
                    fail(SDAG_ERR_UNSUPPORTED, ix.line, ix.col, "index must be iterator +- constant");
                if (pos != q)
                    fail(SDAG_ERR_UNSUPPORTED, ix.line, ix.col,
                         "index position " + std::to_string(q) + " must use iterator '" + P.iters[q] + "'");
                n.off[axis_of_pos(q)] = ix.off;
            }
            return add(n);
        }
        // 1D coefficient array (mixed dimensionality)
        if (r.idx.size() != 1) fail(SDAG_ERR_SEMANTIC, r.line, r.col, "1D array '" + r.s + "' needs one index");
        const RawIdx &ix = r.idx[0];
        int pos = iter_pos(ix.iter);
        if (ix.iter.empty() || pos < 0)
            fail(SDAG_ERR_UNSUPPORTED, ix.line, ix.col, "index must be iterator +- constant");
        int ax = axis_of_pos(pos);
        if (fo.axis >= 0 && fo.axis != ax)
            fail(SDAG_ERR_UNSUPPORTED, ix.line, ix.col, "1D array '" + r.s + "' indexed by two iterators");
        fo.axis = ax;
        fo.role = Role::In;  // a read 1D array (unread ones stay Unused)
        n.kind = Node::Load1;
        n.ref = fo.kind_index;
        n.off[0] = ix.off;
        return add(n);
    }

    void run() {
        n_iter = (int)P.iters.size();
        if (n_iter == 0) fail(SDAG_ERR_SEMANTIC, 1, 1, "no 'iterator' declaration");
        S.name = D.name;
        S.iterators = P.iters;
        S.parameters = P.params;
        S.pragma = D.pragma;
        S.assign = D.assign;
        S.has_call = C != nullptr;
        if (C && C->actuals.size() != D.formals.size())
            fail(SDAG_ERR_SEMANTIC, C->line, C->col,
                 "call passes " + std::to_string(C->actuals.size()) + " arguments, stencil takes " +
                     std::to_string(D.formals.size()));
        int cnt[3] = {0, 0, 0};
        std::set<std::string> seen;
        for (size_t q = 0; q < D.formals.size(); q++) {
            Formal f;
            f.name = D.formals[q];
            if (!seen.insert(f.name).second)
                fail(SDAG_ERR_SEMANTIC, D.line, D.col, "duplicate formal '" + f.name + "'");
            f.actual = C ? C->actuals[q] : f.name;
            auto d = P.decls.find(f.actual);
            if (d == P.decls.end())
                fail(SDAG_ERR_SEMANTIC, C ? C->line : D.line, C ? C->col : D.col,
                     "argument '" + f.actual + "' is not declared");
            size_t nd = d->second.dims.size();
            if (nd == 0) f.kind = ArgKind::Scalar;
            else if ((int)nd == n_iter) f.kind = ArgKind::Array3D;
            else if (nd == 1) f.kind = ArgKind::Array1D;
            else
                fail(SDAG_ERR_UNSUPPORTED, d->second.line, d->second.col,
                     "array '" + f.actual + "' has " + std::to_string(nd) + " dims with " +
                         std::to_string(n_iter) + " iterators");
            f.kind_index = cnt[(int)f.kind]++;
            formal_of[f.name] = (int)S.formals.size();
            S.formals.push_back(f);
        }
        for (auto &rs : D.body) {
            Statement st;
            st.line = rs.line;
            st.declares = rs.declares;
            int rhs = resolve(*rs.rhs);
            // X op= e  ->  X = X op (e)
            if (rs.op != "=") {
                Raw lhs;
                lhs.k = Raw::Name;
                lhs.s = rs.lhs;
                lhs.indexed = rs.lindexed;
                lhs.idx = rs.lidx;
                lhs.line = rs.line;
                lhs.col = rs.col;
                int l = resolve(lhs);
                Node n;
                n.kind = rs.op == "+=" ? Node::Add : rs.op == "-=" ? Node::Sub : rs.op == "*=" ? Node::Mul : Node::Div;
                n.a = l;
                n.b = rhs;
                n.line = rs.line;
                rhs = add(n);
            }
            st.expr = rhs;
            if (rs.lindexed) {
                auto f = formal_of.find(rs.lhs);
                if (f == formal_of.end()) fail(SDAG_ERR_SEMANTIC, rs.line, rs.col, "undeclared array '" + rs.lhs + "'");
                const Formal &fo = S.formals[f->second];
                if (fo.kind != ArgKind::Array3D)
                    fail(SDAG_ERR_UNSUPPORTED, rs.line, rs.col, "only grid arrays may be written");
                if ((int)rs.lidx.size() != n_iter)
                    fail(SDAG_ERR_SEMANTIC, rs.line, rs.col, "wrong number of indices on '" + rs.lhs + "'");
                for (int q = 0; q < n_iter; q++) {
                    if (rs.lidx[q].iter != P.iters[q] || rs.lidx[q].off != 0)
                        fail(SDAG_ERR_UNSUPPORTED, rs.lidx[q].line, rs.lidx[q].col,
                             "array writes must be at offset 0 (shifted writes are a retiming artefact, P:818-823)");
                }
                st.to_array = true;
                st.target = fo.kind_index;
            } else {
                auto f = formal_of.find(rs.lhs);
                if (f != formal_of.end())
                    fail(SDAG_ERR_SEMANTIC, rs.line, rs.col, "cannot assign to argument '" + rs.lhs + "'");
                auto t = temp_of.find(rs.lhs);
                if (rs.declares && t != temp_of.end())
                    fail(SDAG_ERR_SEMANTIC, rs.line, rs.col, "temporary '" + rs.lhs + "' declared twice");
                if (t == temp_of.end()) {
                    temp_of[rs.lhs] = (int)S.temps.size();
                    S.temps.push_back(rs.lhs);
                }
                temp_assigned.insert(rs.lhs);
                st.to_array = false;
                st.target = temp_of[rs.lhs];
            }
            S.stmts.push_back(st);
        }
        if (S.stmts.empty()) fail(SDAG_ERR_SEMANTIC, D.line, D.col, "empty stencil body");
        for (auto &f : S.formals)
            if (f.kind == ArgKind::Array1D && f.axis < 0) f.axis = 2;  // unused 1D array
    }
};

}  // namespace

Stencil parse_spec(const std::string &text) {
    Parser P;
    P.tk = lex(text);
    P.parse();
    if (P.defs.empty()) fail(SDAG_ERR_SEMANTIC, 1, 1, "no 'stencil' function");
    if (P.defs.size() > 1 || P.calls.size() > 1) {
        const int l = P.defs.size() > 1 ? P.defs[1].line : P.calls[1].line;
        const int c = P.defs.size() > 1 ? P.defs[1].col : P.calls[1].col;
        fail(SDAG_ERR_UNSUPPORTED, l, c,
             "multi-stencil program (Fig 3c): plan it with sdag_program_create, one stage per call");
    }
    Stencil S;
    Resolver R(P, P.defs[0], P.calls.empty() ? nullptr : &P.calls[0], S);
    R.run();
    return S;
}

ProgramIR parse_program(const std::string &text) {
    Parser P;
    P.tk = lex(text);
    P.parse();
    if (P.defs.empty()) fail(SDAG_ERR_SEMANTIC, 1, 1, "no 'stencil' function");
    ProgramIR G;
    if (P.calls.empty()) {
        if (P.defs.size() > 1)
            fail(SDAG_ERR_SEMANTIC, P.defs[1].line, P.defs[1].col, "several stencils but no call to order them");
        G.stages.emplace_back();
        Resolver R(P, P.defs[0], nullptr, G.stages.back());
        R.run();
    } else {
        for (const auto &cl : P.calls) {
            G.stages.emplace_back();
            Resolver R(P, *P.def_of(cl.name), &cl, G.stages.back());
            R.run();
        }
    }
    // program arguments: the declared names some stage binds, in declaration order
    std::set<std::string> used;
    for (const auto &st : G.stages)
        for (const auto &f : st.formals) used.insert(f.actual);
    int cnt[3] = {0, 0, 0};
    for (const auto &n : P.decl_order) {
        if (!used.count(n)) continue;
        ProgramArg a;
        a.name = n;
        for (const auto &st : G.stages)
            for (const auto &f : st.formals)
                if (f.actual == n) {
                    a.kind = f.kind;
                    if (f.kind == ArgKind::Array1D) a.axis = f.axis;
                }
        a.kind_index = cnt[int(a.kind)]++;
        G.args.push_back(a);
    }
    for (const auto &st : G.stages) {
        std::vector<int> m;
        for (const auto &f : st.formals)
            for (size_t q = 0; q < G.args.size(); q++)
                if (G.args[q].name == f.actual) m.push_back(int(q));
        G.map.push_back(m);
    }
    return G;
}

}  // namespace sdag
