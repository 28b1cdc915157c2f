// jit.cu -- NEXT-4: arbitrary single-stage stencil DAGs on the
// GPU by run-time code generation.
//
// The paper's framework is a code generator: a DSL spec becomes CUDA source
// (Listing 2).  For DAGs without a hand-written sm_100a body in the
// registry, this file does the same at plan time, B200-style:
//   1. the resolved IR (ir.hpp) is printed as a point body -- one C++
//      expression per statement, fully parenthesised in program order, literals
//      as exact hexadecimal doubles, loads as ring taps g.at(slot,dz,dy,dx),
//      1D arrays as g.s1, scalars as g.s, inout reads-before-write as g.io,
//      reads of an array after its write as the value just computed (the
//      semantics of reading R3 / SURVEY 8(c) c1);
//   2. NVRTC compiles that body into the same z-streaming TMA/LSU skeleton
//      (sweep.cuh, embedded at build time) for a few tile geometries in one
//      program, for sm_100a, into a cubin;
//   3. the cubin is loaded with the driver API in the plan's device context;
//      the plan's candidates are these kernels, launched by plan_launch like
//      the ahead-of-time ones (cuLaunchKernel instead of cudaLaunchKernel).
// Compiled modules are cached per (source, device) for the process lifetime.
// Host-only plans (SDAG_DEVICE_NONE) generate and compile but do not load, so
// the generator and the NVRTC build are testable without a GPU.
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <nvrtc.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <memory>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

#include "plan.hpp"
#include "sweep.cuh"

namespace sdag {

#include "jit_embed.inc"       // kSweepSrc: the text of sweep.cuh
#include "jit_star_embed.inc"  // kStarSrc: the text of star.cuh

// ---------------------------------------------------------------------------
// 1. code generation
// ---------------------------------------------------------------------------

namespace {

std::string num_literal(double v) {
    char buf[64];
    std::snprintf(buf, sizeof buf, "%a", v);  // exact
    return std::string("(") + buf + ")";
}

struct Gen {
    const Plan &p;
    std::vector<bool> written;  // per 3D formal, in program order

    std::string expr(int n) const {
        const Node &x = p.st.nodes[n];
        switch (x.kind) {
        case Node::Num: return num_literal(x.value);
        case Node::Scalar: return "g.s(" + std::to_string(x.ref) + ")";
        case Node::Temp: return "t" + std::to_string(x.ref);
        case Node::Load3: {
            const int f = x.ref;
            if (p.in_slot[f] >= p.n_staged)  // #assign gmem: through L1/L2
                return "g.gm(" + std::to_string(p.in_slot[f]) + ", " + std::to_string(x.off[0]) + ", " +
                       std::to_string(x.off[1]) + ", " + std::to_string(x.off[2]) + ")";
            if (p.in_slot[f] >= 0)
                return "g.at(" + std::to_string(p.in_slot[f]) + ", " + std::to_string(x.off[0]) + ", " +
                       std::to_string(x.off[1]) + ", " + std::to_string(x.off[2]) + ")";
            // a written array, read at offset 0 (analysis rejects shifted reads)
            if (written[f]) return "v" + std::to_string(p.out_slot[f]);
            if (p.io_slot[f] >= 0) return "g.io(" + std::to_string(p.io_slot[f]) + ")";
            throw Error(SDAG_ERR_UNSUPPORTED, "jit: read of an output before it is written");
        }
        case Node::Load1: return "g.s1(" + std::to_string(x.ref) + ", " + std::to_string(x.off[0]) + ")";
        case Node::Neg: return "(-" + expr(x.a) + ")";
        case Node::Add: return "(" + expr(x.a) + " + " + expr(x.b) + ")";
        case Node::Sub: return "(" + expr(x.a) + " - " + expr(x.b) + ")";
        case Node::Mul: return "(" + expr(x.a) + " * " + expr(x.b) + ")";
        case Node::Div: return "(" + expr(x.a) + " / " + expr(x.b) + ")";
        }
        throw Error(SDAG_ERR_UNSUPPORTED, "jit: unknown expression node");
    }
};

}  // namespace

// The body struct for the sweep skeleton (interface: sweep.cuh header).
std::string jit_body_source(const Plan &p, const std::string &sname, int rzr) {
    const int nin = p.n_staged, nout = p.an.n_out + p.an.n_inout, nio = p.an.n_inout, n1 = p.n1();
    std::ostringstream o;
    o << "struct " << sname << " {\n"
      << "    static constexpr int NIN = " << nin << ", NOUT = " << nout << ", NIO = " << nio << ", N1D = " << n1
      << ";\n"
      << "    static constexpr int RZ = " << p.an.radius[0] << ", RY = " << p.an.radius[1]
      << ", RX = " << p.an.radius[2] << ", RZR = " << rzr << ";\n"
      << "    __host__ __device__ static constexpr int axis1d(int a) { return ";
    for (int f = 0; f < n1; f++) o << "a == " << f << " ? " << p.st.formal(ArgKind::Array1D, f).axis << " : ";
    o << "2; }\n"
      << "    template <class G>\n"
      << "    __device__ __forceinline__ static void eval(const G &g, double (&o)[NOUT]) {\n";
    for (size_t t = 0; t < p.st.temps.size(); t++) o << "        double t" << t << " = 0.0;\n";
    for (int m = 0; m < nout; m++) o << "        double v" << m << " = 0.0;\n";
    Gen g{p, std::vector<bool>(p.n3(), false)};
    for (const Statement &s : p.st.stmts) {
        const std::string rhs = g.expr(s.expr);
        if (s.to_array) {
            o << "        v" << p.out_slot[s.target] << " = " << rhs << ";  // line " << s.line << "\n";
            g.written[s.target] = true;
        } else {
            o << "        t" << s.target << " = " << rhs << ";  // line " << s.line << "\n";
        }
    }
    for (int m = 0; m < nout; m++) o << "        o[" << m << "] = v" << m << ";\n";
    o << "    }\n};\n";
    return o.str();
}

// ---------------------------------------------------------------------------
// 1b. star form: a DAG that is LINEAR in its single input, with only on-axis
// taps whose coefficients are mirror-symmetric (and equal for y and z), is
// generated into the hand-written register-queue star kernel (star.cuh)
// instead of the generic skeleton: B = K + c0 A + sum_r cx_r (A(+-r x)) +
// cyz_r (A(+-r y) + A(+-r z)), coefficients any expressions of the scalars.
// ---------------------------------------------------------------------------

namespace {

struct Lin {  // linear form over input taps: tap -> coefficient (C expression of scalars)
    std::map<std::array<int, 3>, std::string> c;
    std::string k;  // constant term ("" = none)
    bool ok = true;
};

std::string cadd(const std::string &a, const std::string &b, char op) {
    if (a.empty()) return op == '+' ? b : "(-" + b + ")";
    if (b.empty()) return a;
    return "(" + a + " " + op + " " + b + ")";
}

Lin lin_of(const Plan &p, int n, const std::vector<Lin> &temps) {
    const Node &x = p.st.nodes[n];
    Lin r;
    auto is_const = [](const Lin &l) { return l.ok && l.c.empty(); };
    switch (x.kind) {
        case Node::Num: r.k = num_literal(x.value); return r;
        case Node::Scalar: r.k = "a.s[" + std::to_string(x.ref) + "]"; return r;
        case Node::Temp: return temps[x.ref];
        case Node::Load3:
            if (p.in_slot[x.ref] != 0 || p.n_staged != 1) r.ok = false;
            else r.c[{x.off[0], x.off[1], x.off[2]}] = "(1.0)";
            return r;
        case Node::Load1: r.ok = false; return r;
        case Node::Neg: {
            Lin a = lin_of(p, x.a, temps);
            for (auto &kv : a.c) kv.second = "(-" + kv.second + ")";
            if (!a.k.empty()) a.k = "(-" + a.k + ")";
            return a;
        }
        case Node::Add:
        case Node::Sub: {
            const char op = x.kind == Node::Add ? '+' : '-';
            Lin a = lin_of(p, x.a, temps), b = lin_of(p, x.b, temps);
            if (!a.ok || !b.ok) { r.ok = false; return r; }
            r = a;
            for (auto &kv : b.c) r.c[kv.first] = cadd(r.c.count(kv.first) ? r.c[kv.first] : "", kv.second, op);
            if (!b.k.empty()) r.k = cadd(r.k, b.k, op);
            return r;
        }
        case Node::Mul:
        case Node::Div: {
            Lin a = lin_of(p, x.a, temps), b = lin_of(p, x.b, temps);
            if (!a.ok || !b.ok) { r.ok = false; return r; }
            const char op = x.kind == Node::Mul ? '*' : '/';
            if (is_const(b)) {  // (linear) op const
                for (auto &kv : a.c) kv.second = "(" + kv.second + " " + op + " " + b.k + ")";
                if (!a.k.empty()) a.k = "(" + a.k + " " + op + " " + b.k + ")";
                return a;
            }
            if (op == '*' && is_const(a)) {
                for (auto &kv : b.c) kv.second = "(" + a.k + " * " + kv.second + ")";
                if (!b.k.empty()) b.k = "(" + a.k + " * " + b.k + ")";
                return b;
            }
            r.ok = false;  // product or quotient of taps: not linear
            return r;
        }
    }
    r.ok = false;
    return r;
}

}  // namespace

// Box form: linear in the one input, taps within the 3x3x3 box, the
// coefficient of a tap depending only on its class (centre / face / edge /
// corner, by the number of nonzero offsets) -> the retimed, folded box27
// kernel (FORM 2).  Weights w0..w3 (expressions of the scalars) are evaluated
// on the host at each launch.  Returns false when the DAG is not in box form.
bool jit_box_form(const Plan &p, std::vector<std::string> &w) {
    if (p.an.n_in != 1 || p.n_staged != 1 || p.an.n_out != 1 || p.an.n_inout != 0 || p.n1() != 0) return false;
    if (p.an.radius[0] != 1 || p.an.radius[1] != 1 || p.an.radius[2] != 1) return false;
    std::vector<Lin> temps(p.st.temps.size());
    Lin out;
    int writes = 0;
    for (const Statement &st : p.st.stmts) {
        Lin v = lin_of(p, st.expr, temps);
        if (!v.ok) return false;
        if (st.to_array) {
            out = v;
            writes++;
        } else {
            temps[st.target] = v;
        }
    }
    if (writes != 1 || !out.k.empty()) return false;
    std::string cls[4];
    bool seen[4] = {false, false, false, false};
    for (int dz = -1; dz <= 1; dz++)
        for (int dy = -1; dy <= 1; dy++)
            for (int dx = -1; dx <= 1; dx++) {
                const int c = (dz != 0) + (dy != 0) + (dx != 0);
                auto it = out.c.find({dz, dy, dx});
                const std::string v = it == out.c.end() ? "(0.0)" : it->second;
                if (!seen[c]) {
                    cls[c] = v;
                    seen[c] = true;
                } else if (cls[c] != v) {
                    return false;
                }
            }
    w.assign(cls, cls + 4);
    return true;
}

namespace {
struct CoefEval {  // recursive descent over the generated coefficient text
    const char *q;
    const double *s;
    int ns;
    void ws() {
        while (*q == ' ') q++;
    }
    double factor() {
        ws();
        if (*q == '(') {
            q++;
            const double v = expr();
            ws();
            if (*q != ')') throw Error(SDAG_ERR_INVALID_ARG, "coefficient: ')' expected");
            q++;
            return v;
        }
        if (*q == '-') {
            q++;
            return -factor();
        }
        if (std::strncmp(q, "a.s[", 4) == 0) {
            q += 4;
            const int i = int(std::strtol(q, const_cast<char **>(&q), 10));
            if (*q != ']' || i < 0 || i >= ns) throw Error(SDAG_ERR_INVALID_ARG, "coefficient: bad scalar index");
            q++;
            return s[i];
        }
        char *end = nullptr;
        const double v = std::strtod(q, &end);
        if (end == q) throw Error(SDAG_ERR_INVALID_ARG, "coefficient: number expected");
        q = end;
        return v;
    }
    double term() {
        double v = factor();
        for (;;) {
            ws();
            if (*q == '*') q++, v = v * factor();
            else if (*q == '/') q++, v = v / factor();
            else return v;
        }
    }
    double expr() {
        double v = term();
        for (;;) {
            ws();
            if (*q == '+') q++, v = v + term();
            else if (*q == '-') q++, v = v - term();
            else return v;
        }
    }
};
}  // namespace

double jit_eval_coef(const std::string &e, const double *s, int ns) {
    CoefEval c{e.c_str(), s, ns};
    return c.expr();
}

// The star body for star.cuh, or "" when the DAG is not in star form.
std::string jit_star_body(const Plan &p, int *R_out) {
    if (p.an.n_in != 1 || p.n_staged != 1 || p.an.n_out != 1 || p.an.n_inout != 0 || p.n1() != 0) return "";
    std::vector<Lin> temps(p.st.temps.size());
    Lin out;
    int writes = 0;
    for (const Statement &st : p.st.stmts) {
        Lin v = lin_of(p, st.expr, temps);
        if (!v.ok) return "";
        if (st.to_array) {
            out = v;
            writes++;
        } else {
            temps[st.target] = v;
        }
    }
    if (writes != 1) return "";  // accumulating writes read the output: not this form
    int R = 0;
    for (auto &kv : out.c) {
        const auto &t = kv.first;
        const int nz = (t[0] != 0) + (t[1] != 0) + (t[2] != 0);
        if (nz > 1) return "";  // off-axis tap
        R = std::max({R, std::abs(t[0]), std::abs(t[1]), std::abs(t[2])});
    }
    if (R < 1 || R > 4) return "";
    auto coef = [&](int dz, int dy, int dx) {
        auto it = out.c.find({dz, dy, dx});
        return it == out.c.end() ? std::string("(0.0)") : it->second;
    };
    std::ostringstream cx, cyz, cz;
    bool split = false;
    for (int r = 1; r <= R; r++) {
        const std::string xp = coef(0, 0, r), xm = coef(0, 0, -r), yp = coef(0, r, 0), ym = coef(0, -r, 0),
                          zp = coef(r, 0, 0), zm = coef(-r, 0, 0);
        if (xp != xm || yp != ym || zp != zm) return "";  // not mirror-symmetric
        if (yp != zp) split = true;                      // distinct y and z coefficients
        cx << "        case " << r << ": return " << xp << ";\n";
        cyz << "        case " << r << ": return " << yp << ";\n";
        cz << "        case " << r << ": return " << zp << ";\n";
    }
    *R_out = R;
    std::ostringstream o;
    o << "struct JitStar {\n"
      << "    static constexpr int R = " << R << ", NIN = 1, NOUT = 1, NIO = 0, N1D = 0, RZ = " << R << ", RY = " << R
      << ", RX = " << R << ", RZR = " << R << ";\n"
      << "    static constexpr bool SPLIT_YZ = " << (split ? "true" : "false") << ";\n"
      << "    __host__ __device__ static constexpr int axis1d(int) { return 2; }\n"
      << "    __device__ __forceinline__ static double cx(const SweepArgs &a, int r) {\n"
      << "        switch (r) {\n" << cx.str() << "        default: return 0.0;\n        }\n    }\n"
      << "    __device__ __forceinline__ static double cyz(const SweepArgs &a, int r) {\n"
      << "        switch (r) {\n" << cyz.str() << "        default: return 0.0;\n        }\n    }\n"
      << "    __device__ __forceinline__ static double cz(const SweepArgs &a, int r) {\n"
      << "        switch (r) {\n" << cz.str() << "        default: return 0.0;\n        }\n    }\n"
      << "    __device__ __forceinline__ static void yz(double &acc, const SweepArgs &a, int r, double s) {\n"
      << "        acc = fma(cyz(a, r), s, acc);\n    }\n"
      << "    __device__ __forceinline__ static void y(double &acc, const SweepArgs &a, int r, double s) {\n"
      << "        acc = fma(cyz(a, r), s, acc);\n    }\n"
      << "    __device__ __forceinline__ static void z(double &acc, const SweepArgs &a, int r, double s) {\n"
      << "        acc = fma(cz(a, r), s, acc);\n    }\n"
      << "    __device__ __forceinline__ static void x(double &acc, const SweepArgs &a, int r, double s) {\n"
      << "        acc = fma(cx(a, r), s, acc);\n    }\n"
      << "    __device__ __forceinline__ static double finish(double acc, const SweepArgs &a, double ctr) {\n"
      << "        return fma(" << coef(0, 0, 0) << ", ctr, acc)" << (out.k.empty() ? "" : " + " + out.k) << ";\n"
      << "    }\n};\n";
    return o.str();
}

// ---------------------------------------------------------------------------
// 2. NVRTC (dlopen'ed, like NCCL in dist.cpp: no link-time dependency)
// ---------------------------------------------------------------------------

namespace {

struct Nvrtc {
    decltype(&nvrtcCreateProgram) create = nullptr;
    decltype(&nvrtcAddNameExpression) add_name = nullptr;
    decltype(&nvrtcCompileProgram) compile = nullptr;
    decltype(&nvrtcGetProgramLogSize) log_size = nullptr;
    decltype(&nvrtcGetProgramLog) log = nullptr;
    decltype(&nvrtcGetCUBINSize) cubin_size = nullptr;
    decltype(&nvrtcGetCUBIN) cubin = nullptr;
    decltype(&nvrtcGetLoweredName) lowered = nullptr;
    decltype(&nvrtcDestroyProgram) destroy = nullptr;
    decltype(&nvrtcGetErrorString) errstr = nullptr;
};

const Nvrtc &nvrtc() {
    static Nvrtc n = [] {
        Nvrtc r;
        void *h = nullptr;
        for (const char *name : {"libnvrtc.so.12", "libnvrtc.so", "/usr/local/cuda/lib64/libnvrtc.so.12"})
            if ((h = dlopen(name, RTLD_NOW | RTLD_LOCAL))) break;
        if (!h) throw Error(SDAG_ERR_UNSUPPORTED, "jit: libnvrtc.so.12 not found (needed for unregistered DAGs)");
        auto sym = [&](const char *s) {
            void *f = dlsym(h, s);
            if (!f) throw Error(SDAG_ERR_UNSUPPORTED, std::string("jit: nvrtc symbol missing: ") + s);
            return f;
        };
        r.create = reinterpret_cast<decltype(r.create)>(sym("nvrtcCreateProgram"));
        r.add_name = reinterpret_cast<decltype(r.add_name)>(sym("nvrtcAddNameExpression"));
        r.compile = reinterpret_cast<decltype(r.compile)>(sym("nvrtcCompileProgram"));
        r.log_size = reinterpret_cast<decltype(r.log_size)>(sym("nvrtcGetProgramLogSize"));
        r.log = reinterpret_cast<decltype(r.log)>(sym("nvrtcGetProgramLog"));
        r.cubin_size = reinterpret_cast<decltype(r.cubin_size)>(sym("nvrtcGetCUBINSize"));
        r.cubin = reinterpret_cast<decltype(r.cubin)>(sym("nvrtcGetCUBIN"));
        r.lowered = reinterpret_cast<decltype(r.lowered)>(sym("nvrtcGetLoweredName"));
        r.destroy = reinterpret_cast<decltype(r.destroy)>(sym("nvrtcDestroyProgram"));
        r.errstr = reinterpret_cast<decltype(r.errstr)>(sym("nvrtcGetErrorString"));
        return r;
    }();
    return n;
}

// driver entry points through the runtime (libsdag links cudart statically)
template <class F>
F drv(const char *name) {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    check_cuda(cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q), name);
    if (!p || q != cudaDriverEntryPointSuccess) throw Error(SDAG_ERR_CUDA, std::string(name) + " not available");
    return reinterpret_cast<F>(p);
}

void check_cu(CUresult r, const char *what) {
    if (r != CUDA_SUCCESS) throw Error(SDAG_ERR_CUDA, std::string(what) + " failed (CUresult " + std::to_string(r) + ")");
}

struct Compiled {
    std::string cubin;
    std::vector<std::string> lowered;  // per name expression
    std::string log;
};

Compiled nvrtc_build(const std::string &src, const std::vector<std::string> &names, int maxrreg = 0,
                      bool strict = false) {
    const Nvrtc &N = nvrtc();
    nvrtcProgram prog;
    auto ck = [&](nvrtcResult r, const char *what) {
        if (r != NVRTC_SUCCESS) throw Error(SDAG_ERR_CUDA, std::string("jit: ") + what + ": " + N.errstr(r));
    };
    ck(N.create(&prog, src.c_str(), "sdag_jit.cu", 0, nullptr, nullptr), "nvrtcCreateProgram");
    Compiled c;
    try {
        for (const auto &n : names) ck(N.add_name(prog, n.c_str()), "nvrtcAddNameExpression");
        std::vector<const char *> opts = {"-arch=sm_100a", "-std=c++17", "-default-device",
                                          strict ? "--fmad=false" : "--fmad=true", "-lineinfo",
                                          "--extra-device-vectorization"};
        const std::string rr = "--maxrregcount=" + std::to_string(maxrreg);
        if (maxrreg > 0) opts.push_back(rr.c_str());  // occupancy t: register rationing
        const nvrtcResult rc = N.compile(prog, int(opts.size()), opts.data());
        size_t ls = 0;
        N.log_size(prog, &ls);
        c.log.assign(ls, '\0');
        if (ls) N.log(prog, &c.log[0]);
        if (rc != NVRTC_SUCCESS)
            throw Error(SDAG_ERR_UNSUPPORTED, "jit: NVRTC compile failed: " + std::string(N.errstr(rc)) + "\n" + c.log);
        size_t cs = 0;
        ck(N.cubin_size(prog, &cs), "nvrtcGetCUBINSize");
        c.cubin.assign(cs, '\0');
        ck(N.cubin(prog, &c.cubin[0]), "nvrtcGetCUBIN");
        for (const auto &n : names) {
            const char *l = nullptr;
            ck(N.lowered(prog, n.c_str(), &l), "nvrtcGetLoweredName");
            c.lowered.push_back(l);
        }
    } catch (...) {
        N.destroy(&prog);
        throw;
    }
    N.destroy(&prog);
    return c;
}

struct Module {
    CUmodule mod = nullptr;
    std::vector<CUfunction> fns;
};

std::mutex g_jit_mu;
std::map<std::string, Compiled> g_compiled;            // source -> cubin
std::map<std::pair<std::string, int>, Module> g_mods;  // (source, device) -> module

struct Geom {
    int tx, ty, ux, uy, pf;
};

}  // namespace

// ---------------------------------------------------------------------------
// 3. plan integration
// ---------------------------------------------------------------------------

// Fill p->jit_descs / p->cands with NVRTC-compiled skeleton kernels for the
// plan's DAG.  Throws UNSUPPORTED when the DAG exceeds the skeleton's limits.
void jit_build_candidates(Plan *p) {
    using namespace dev;
    const int nin_all = p->an.n_in, nout = p->an.n_out + p->an.n_inout, nio = p->an.n_inout, n1 = p->n1();
    if (p->n_staged < 1 || nin_all > MAXIN || nout > MAXOUT || nio > MAXIO || n1 > MAX1D || p->ns() > MAXS)
        throw Error(SDAG_ERR_UNSUPPORTED,
                    "jit: DAG outside the sweep skeleton's limits (1.." + std::to_string(MAXIN) + " inputs, <= " +
                        std::to_string(MAXOUT) + " outputs, <= " + std::to_string(MAXIO) + " inouts, <= " +
                        std::to_string(MAX1D) + " 1D arrays, <= " + std::to_string(MAXS) + " scalars)");
    const int RZ = p->an.radius[0], RY = p->an.radius[1], RX = p->an.radius[2];
    int nin = p->n_staged;

    // tile geometries, preference order (the generic skeleton's best shapes on
    // the registered DAGs: tools/perf_sweep.py); smem decides RZR
    std::vector<Geom> geoms = {{32, 16, 1, 2, 1}, {64, 8, 1, 1, 1}, {16, 16, 1, 1, 1}};
    // the spec's "#pragma ... block (bx,by) unroll j=u": the user's
    // thread block and unroll factors become the first candidate geometry
    // (tile = block x unroll per axis)
    const Pragma &pr = p->st.pragma;
    if (pr.block[0] > 0 && p->st.iterators.size() == 3) {
        auto un = [&](int axis) {
            auto it = pr.unroll.find(p->st.iterators[axis]);
            return it == pr.unroll.end() ? 1 : it->second;
        };
        const int ux = un(2), uy = un(1), bx = pr.block[0], by = pr.block[1] > 0 ? pr.block[1] : 1;
        const Geom g{bx * ux, by * uy, ux, uy, 1};
        if (ux >= 1 && uy >= 1 && ux * uy <= 16 && bx * by >= 32 && bx * by <= 1024) {
            geoms.erase(std::remove_if(geoms.begin(), geoms.end(),
                                       [&](const Geom &h) {
                                           return h.tx == g.tx && h.ty == g.ty && h.ux == g.ux && h.uy == g.uy;
                                       }),
                        geoms.end());
            geoms.insert(geoms.begin(), g);
        }
    }
    struct Cand {
        Geom g;
        int rzr;
        bool tma;
        int smem;
        std::string name;
    };
    std::vector<Cand> cs;
    bool need_r0 = false, need_full = false;
    // z-queue variants (sweep.cuh sdag_sweepq): on-axis z-taps from registers,
    // the ring only as deep as the off-axis taps need
    int rz_off = 0;
    for (const Node &n : p->st.nodes)
        if (n.kind == Node::Load3 && (n.off[1] != 0 || n.off[2] != 0) && p->in_slot[n.ref] >= 0 &&
            p->in_slot[n.ref] < p->n_staged)
            rz_off = std::max(rz_off, std::abs(n.off[0]));
    struct CandQ {
        Geom g;
        bool tma;
        int smem;
        std::string name;
    };
    std::vector<CandQ> cq;

    // "#pragma ... occupancy t": t x 2048 threads must be resident per
    // SM.  Registers are rationed with --maxrregcount; while shared memory still
    // prevents it for the first geometry, the staged input with the fewest
    // accesses is demoted to global memory (read through L1/L2, as #assign gmem),
    // until the ring fits or one input is left staged.
    int maxrreg = 0;
    int nstage = nin;
    if (pr.occupancy > 0) {
        const Geom &g0 = geoms[0];
        const int thr = (g0.tx / g0.ux) * (g0.ty / g0.uy);
        const int target = std::max(thr, int(pr.occupancy * 2048.0 + 0.5));
        maxrreg = std::max(32, std::min(255, (65536 / target) / 8 * 8));
        const int plane_al = (((g0.tx + 2 * RX) * (g0.ty + 2 * RY) * 8 + 127) / 128) * 128 / 8;
        auto resident = [&](int ns_in) {
            const int smem = (2 * RZ + 1 + g0.pf) * ns_in * plane_al * 8 + (2 * RZ + 1 + g0.pf) * 8;
            const int by_smem = smem > 0 ? (228 * 1024) / (smem + 1024) : 32;
            return std::min(2048 / thr, by_smem) * thr;
        };
        std::vector<int> acc(p->n3(), 0);  // accesses per 3D formal
        for (const Node &n : p->st.nodes)
            if (n.kind == Node::Load3) acc[n.ref]++;
        while (nstage > 1 && resident(nstage) < target) {
            int victim = -1;
            for (int f = 0; f < p->n3(); f++)
                if (p->in_slot[f] >= 0 && p->in_slot[f] < nstage &&
                    (victim < 0 || acc[f] < acc[victim]))
                    victim = f;
            // move the victim to the last staged slot, then shrink the staged range
            const int last = nstage - 1, vs = p->in_slot[victim];
            for (int f = 0; f < p->n3(); f++)
                if (p->in_slot[f] == last) p->in_slot[f] = vs;
            p->in_slot[victim] = last;
            nstage--;
        }
        p->n_staged = nstage;
        p->jit_maxrreg = maxrreg;
        nin = nstage;
    }
    if (RZ > 0) {
        for (const Geom &g : geoms) {
            const int px = g.tx + 2 * RX, py = g.ty + 2 * RY;
            if (px > 256 || py > 256) continue;
            if (nin * (2 * RZ + 1) * g.ux * g.uy > 48) continue;  // queue registers
            const int plane_al = ((px * py * 8 + 127) / 128) * 128 / 8;
            const int ns = RZ + rz_off + 1 + g.pf;
            const int smem = ns * nin * plane_al * 8 + ns * 8;
            if (smem > 227 * 1024) continue;
            for (bool tma : {true, false}) cq.push_back({g, tma, smem, ""});
        }
    }
    for (const Geom &g : geoms) {
        const int px = g.tx + 2 * RX, py = g.ty + 2 * RY;
        if (px > 256 || py > 256) continue;
        const int plane_al = ((px * py * 8 + 127) / 128) * 128 / 8;
        for (int rzr : {RZ, 0}) {
            const int ns = 2 * rzr + 1 + g.pf;
            const int smem = ns * nin * plane_al * 8 + ns * 8;
            if (smem > 227 * 1024) continue;
            (rzr == RZ ? need_full : need_r0) = true;
            for (bool tma : {true, false}) cs.push_back({g, rzr, tma, smem, ""});
            break;
        }
    }
    if (cs.empty()) throw Error(SDAG_ERR_UNSUPPORTED, "jit: no tile geometry fits 227 KB of shared memory");

    std::ostringstream src;
    src << "// generated by sdag jit.cpp for stencil '" << p->st.name << "'"
        << (maxrreg ? " (--maxrregcount=" + std::to_string(maxrreg) + ")" : std::string()) << "\n" << kSweepSrc << "\n"
        << "namespace sdag {\nnamespace dev {\n";
    if (need_full) src << jit_body_source(*p, "JitBody", RZ);
    if (need_r0 && RZ > 0) src << jit_body_source(*p, "JitBodyR0", 0);
    if (need_r0 && RZ == 0 && !need_full) src << jit_body_source(*p, "JitBody", 0);
    if (!cq.empty()) src << jit_body_source(*p, "JitBodyQ", rz_off);
    // star form (linear, on-axis, mirror-symmetric): the hand-written star kernel
    int Rstar = 0;
    const std::string star_body = (p->st.pragma.block[0] > 0 || p->st.pragma.occupancy > 0 || p->jit_strict)
                                      ? std::string()  // user guidance / strict order: the generic skeleton
                                      : jit_star_body(*p, &Rstar);
    struct CandS {
        int tx, ty, uy, pf, unr;
        std::string name;
        int smem, threads;
    };
    std::vector<CandS> cst;
    p->jit_star_src = star_body;
    p->box_w.clear();  // (a radius-1 star is also in box form: box kernels + temporal fusion, star kernels too)
    if (!(p->st.pragma.block[0] > 0 || p->st.pragma.occupancy > 0 || p->jit_strict)) jit_box_form(*p, p->box_w);
    if (!star_body.empty()) {
        src << "}  // namespace dev\n}  // namespace sdag\n" << kStarSrc << "\nnamespace sdag {\nnamespace dev {\n"
            << star_body;
        // the registered star geometries (lap25 / jacobi7 measured picks, DESIGN 6.3)
        // (radius <= 2: Jacobi's 64x16 first; wider radii: the Laplacian's 32x32)
        const int big[2][5] = {{32, 32, 4, 3, 2}, {64, 16, 2, 3, 1}}, small[2][5] = {{64, 16, 2, 3, 1}, {32, 32, 4, 3, 2}};
        for (const auto &g : (Rstar <= 2 ? small : big)) {
            const int ML = Rstar + (Rstar % 2), px = g[0] + 2 * ML, py = g[1] + 2 * Rstar;
            const int plane_al = ((px * py * 8 + 127) / 128) * 128 / 8, ns = Rstar + 1 + g[3];
            const int smem = ns * plane_al * 8 + 2 * ns * 8;
            if (px > 256 || py > 256 || smem > 227 * 1024) continue;
            char buf[96];
            std::snprintf(buf, sizeof buf, "jitstar_tma_%dx%d_u2x%d_pf%d%s", g[0], g[1], g[2], g[3],
                          g[4] > 1 ? "_z2" : "");
            cst.push_back({g[0], g[1], g[2], g[3], g[4], buf, smem, (g[0] / 2) * (g[1] / g[2])});
        }
    }
    src << "}  // namespace dev\n}  // namespace sdag\n";
    std::vector<std::string> names;
    for (Cand &c : cs) {
        const char *body = (c.rzr == RZ) ? "JitBody" : "JitBodyR0";
        char buf[160];
        std::snprintf(buf, sizeof buf, "sdag::dev::sdag_sweep<sdag::dev::%s, %d, %d, %d, %d, %d, %s>", body, c.g.tx,
                      c.g.ty, c.g.ux, c.g.uy, c.g.pf, c.tma ? "true" : "false");
        names.push_back(buf);
        std::snprintf(buf, sizeof buf, "jit_%s_%dx%d_u%dx%d_pf%d%s%s", c.tma ? "tma" : "lsu", c.g.tx, c.g.ty, c.g.ux,
                      c.g.uy, c.g.pf, (c.rzr == RZ) ? "" : "_r0", p->jit_strict ? "_strict" : "");
        c.name = buf;
    }
    for (CandQ &c : cq) {
        char buf[160];
        std::snprintf(buf, sizeof buf, "sdag::dev::sdag_sweepq<sdag::dev::JitBodyQ, %d, %d, %d, %d, %d, %s>", c.g.tx,
                      c.g.ty, c.g.ux, c.g.uy, c.g.pf, c.tma ? "true" : "false");
        names.push_back(buf);
        std::snprintf(buf, sizeof buf, "jitq_%s_%dx%d_u%dx%d_pf%d%s", c.tma ? "tma" : "lsu", c.g.tx, c.g.ty, c.g.ux,
                      c.g.uy, c.g.pf, p->jit_strict ? "_strict" : "");
        c.name = buf;
    }
    for (CandS &c : cst) {
        char buf[200];
        std::snprintf(buf, sizeof buf, "sdag::dev::sdag_star<sdag::dev::JitStar, %d, %d, %d, %d, true, 0, 1, %d>", c.tx,
                      c.ty, c.uy, c.pf, c.unr);
        names.push_back(buf);
    }
    const std::string key = src.str();

    std::lock_guard<std::mutex> lk(g_jit_mu);
    // compile (cached by source and register cap) and load on the plan's device
    auto build = [&](int cap) {
        const std::string ck = (cap ? key + "// --maxrregcount=" + std::to_string(cap) + "\n" : key) +
                               (p->jit_strict ? "// --fmad=false\n" : "");
        auto it = g_compiled.find(ck);
        if (it == g_compiled.end()) it = g_compiled.emplace(ck, nvrtc_build(key, names, cap, p->jit_strict)).first;
        const Compiled &cc = it->second;
        std::vector<CUfunction> fns(names.size(), nullptr);
        if (p->host_only) return fns;
        auto mk = std::make_pair(ck, p->device);
        auto mt = g_mods.find(mk);
        if (mt == g_mods.end()) {
            int prev = -1;
            check_cuda(cudaGetDevice(&prev), "cudaGetDevice");
            check_cuda(cudaSetDevice(p->device), "cudaSetDevice");
            check_cuda(cudaFree(nullptr), "context init");  // make the primary context current
            using LoadT = decltype(&cuModuleLoadData);
            using GetT = decltype(&cuModuleGetFunction);
            Module m;
            CUresult r = drv<LoadT>("cuModuleLoadData")(&m.mod, cc.cubin.data());
            if (r == CUDA_SUCCESS)
                for (const auto &l : cc.lowered) {
                    CUfunction f = nullptr;
                    r = drv<GetT>("cuModuleGetFunction")(&f, m.mod, l.c_str());
                    if (r != CUDA_SUCCESS) break;
                    m.fns.push_back(f);
                }
            cudaSetDevice(prev);
            check_cu(r, "jit: cuModuleLoadData/cuModuleGetFunction");
            mt = g_mods.emplace(mk, m).first;
        }
        return mt->second.fns;
    };
    p->jit_source = key;
    std::vector<CUfunction> fns = build(maxrreg);
    for (size_t q = 0; q < cs.size(); q++) {
        const Cand &c = cs[q];
        auto d = std::make_unique<KernelDesc>();
        d->dag = "(jit)";
        d->variant = c.name;
        d->fn = nullptr;
        d->cufn = fns[q];
        d->threads = (c.g.tx / c.g.ux) * (c.g.ty / c.g.uy);
        d->smem = c.smem;
        d->tx = c.g.tx;
        d->ty = c.g.ty;
        d->ux = c.g.ux;
        d->uy = c.g.uy;
        d->pf = c.g.pf;
        d->tma = c.tma;
        d->nin = nin;
        d->nout = nout;
        d->nio = nio;
        d->n1d = n1;
        d->rz = RZ;
        d->ry = RY;
        d->rx = RX;
        d->rzr = c.rzr;
        d->prio = int(q / 2) + (c.tma ? 0 : 100);
        p->jit_descs.push_back(std::move(d));
    }
    for (size_t q = 0; q < cq.size(); q++) {
        const CandQ &c = cq[q];
        auto d = std::make_unique<KernelDesc>();
        d->dag = "(jit)";
        d->variant = c.name;
        d->fn = nullptr;
        d->cufn = fns[cs.size() + q];
        d->threads = (c.g.tx / c.g.ux) * (c.g.ty / c.g.uy);
        d->smem = c.smem;
        d->tx = c.g.tx;
        d->ty = c.g.ty;
        d->ux = c.g.ux;
        d->uy = c.g.uy;
        d->pf = c.g.pf;
        d->tma = c.tma;
        d->nin = nin;
        d->nout = nout;
        d->nio = nio;
        d->n1d = n1;
        d->rz = RZ;
        d->ry = RY;
        d->rx = RX;
        d->rzr = rz_off;
        d->prio = -10 + int(q / 2) + (c.tma ? 0 : 100);  // preferred: 1.35x (lap25), 1.1x (27-pt) over the ring-only skeleton
        p->jit_descs.push_back(std::move(d));
    }

    for (size_t q = 0; q < cst.size(); q++) {
        const CandS &c = cst[q];
        auto d = std::make_unique<KernelDesc>();
        d->dag = "(jit)";
        d->variant = c.name;
        d->fn = nullptr;
        d->cufn = fns[cs.size() + cq.size() + q];
        d->threads = c.threads;
        d->smem = c.smem;
        d->tx = c.tx;
        d->ty = c.ty;
        d->ux = 2;
        d->uy = c.uy;
        d->pf = c.pf;
        d->tma = true;
        d->nin = 1;
        d->nout = 1;
        d->rz = Rstar;
        d->ry = Rstar;
        d->rx = Rstar + (Rstar % 2);  // TMA box margin (star.cuh ML)
        d->rzr = Rstar;
        d->prio = -50 + int(q);  // the register-queue star kernel first (before box kernels: radius-1 stars)
        p->jit_descs.push_back(std::move(d));
    }

    // register-cap stepping: with tune=1 the TMA candidates are
    // also compiled at 128 and 64 registers per thread; the spill-free ones
    // (no local memory) join the measured candidates as "<variant>_rr<cap>"
    if (p->tune && !p->host_only && maxrreg == 0) {
        using AttrT = decltype(&cuFuncGetAttribute);
        const size_t base = p->jit_descs.size();
        for (int cap : {128, 64}) {
            const std::vector<CUfunction> cf = build(cap);
            for (size_t q = 0; q < base; q++) {
                const KernelDesc &k0 = *p->jit_descs[q];
                if (!k0.tma) continue;
                const size_t fi = q;  // descriptors were created in name order
                int local = 0;
                check_cu(drv<AttrT>("cuFuncGetAttribute")(&local, CU_FUNC_ATTRIBUTE_LOCAL_SIZE_BYTES, cf[fi]),
                         "jit: cuFuncGetAttribute");
                if (local > 0) continue;  // spills: not explored
                auto d = std::make_unique<KernelDesc>(k0);
                d->variant += "_rr" + std::to_string(cap);
                d->cufn = cf[fi];
                d->prio += 50;
                p->jit_descs.push_back(std::move(d));
            }
        }
    }
}

// launch / occupancy of a JIT kernel (driver API)
void jit_launch(const KernelDesc &k, dim3 grid, void **args, cudaStream_t stream) {
    using AttrT = decltype(&cuFuncSetAttribute);
    using LaunchT = decltype(&cuLaunchKernel);
    static AttrT set_attr = drv<AttrT>("cuFuncSetAttribute");
    static LaunchT launch = drv<LaunchT>("cuLaunchKernel");
    CUfunction f = static_cast<CUfunction>(k.cufn);
    check_cu(set_attr(f, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, k.smem), "jit: cuFuncSetAttribute");
    check_cu(launch(f, grid.x, grid.y, grid.z, k.threads, 1, 1, unsigned(k.smem), reinterpret_cast<CUstream>(stream),
                    args, nullptr),
             "jit: cuLaunchKernel");
}

int jit_occupancy(const KernelDesc &k) {
    using OccT = decltype(&cuOccupancyMaxActiveBlocksPerMultiprocessor);
    static OccT occ = drv<OccT>("cuOccupancyMaxActiveBlocksPerMultiprocessor");
    int n = 0;
    if (occ(&n, static_cast<CUfunction>(k.cufn), k.threads, size_t(k.smem)) != CUDA_SUCCESS) return 0;
    return n;
}

}  // namespace sdag
