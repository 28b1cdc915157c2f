// program.cpp -- multi-stencil programs (Fig 3c,
// P:1349-1368): several `stencil` definitions and calls in sequence.
//
// Each call is a stage planned on its own (registered sm_100a kernel or the
// NVRTC-generated one, a3), and the stages run in call order on one stream as
// separate sweeps: a later stage reads what earlier stages wrote, at any
// offset, because every sweep completes before the next starts (stream
// order).  This is the paper's "kernel composition" without the
// cross-stage fusion -- fused stages need a recomputation halo,
// which is the next step.  The program's arguments are its declared arrays
// and scalars in declaration order (the generated host function takes the
// declarations); a stage's formal q is program argument map[s][q].
#include <cuda_runtime.h>

#include <algorithm>
#include <memory>
#include <string>
#include <vector>

#include "plan.hpp"

namespace sdag {

const ProgramArg &Program::arg(ArgKind k, int idx) const {
    for (auto &a : ir.args)
        if (a.kind == k && a.kind_index == idx) return a;
    throw Error(SDAG_ERR_INVALID_ARG, "argument index out of range");
}

Program::~Program() {
    for (sdag_plan_s *h : handles) delete h;
}

Program *program_create(const std::string &spec, const int64_t dims[3], const sdag_plan_opts &o) {
    std::unique_ptr<Program> g(new Program());
    g->ir = parse_program(spec);
    for (size_t s = 0; s < g->ir.stages.size(); s++) {
        g->stages.emplace_back(plan_create_from(g->ir.stages[s], dims, o));
        g->handles.push_back(new sdag_plan_s{g->stages.back().get()});
        log_plan(g->stages.back().get(), ("program stage " + std::to_string(s)).c_str());
    }
    // program-level roles of the 3D arrays, in call order: read before any
    // stage wrote it -> In (InOut once written later); first touched by a
    // write -> Out (an intermediate read by later stages is still caller memory)
    for (size_t s = 0; s < g->stages.size(); s++) {
        const Plan &p = *g->stages[s];
        for (size_t q = 0; q < p.st.formals.size(); q++) {
            const Formal &f = p.st.formals[q];
            if (f.kind != ArgKind::Array3D || f.role == Role::Unused) continue;
            ProgramArg &a = g->ir.args[g->ir.map[s][q]];
            const bool reads = f.role == Role::In || f.role == Role::InOut;
            const bool writes = f.role == Role::Out || f.role == Role::InOut;
            if (a.role == Role::Unused) a.role = reads ? (writes ? Role::InOut : Role::In) : Role::Out;
            else if (a.role == Role::In && writes) a.role = Role::InOut;
        }
    }
    return g.release();
}

void program_apply(Program *g, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns,
                   int batch, cudaStream_t stream) {
    if (n3 != g->n_of(ArgKind::Array3D) || n1 != g->n_of(ArgKind::Array1D) || ns != g->n_of(ArgKind::Scalar))
        throw Error(SDAG_ERR_INVALID_ARG, "expected " + std::to_string(g->n_of(ArgKind::Array3D)) + " grid arrays, " +
                                              std::to_string(g->n_of(ArgKind::Array1D)) + " 1D arrays and " +
                                              std::to_string(g->n_of(ArgKind::Scalar)) + " scalars");
    if ((n3 && !a3) || (n1 && !a1) || (ns && !s)) throw Error(SDAG_ERR_INVALID_ARG, "null argument array");
    NvtxRange nr("sdag_program_apply " + std::to_string(g->stages.size()) + " stages");
    // bind every stage first (all validation before anything is enqueued)
    struct Bound {
        std::vector<double *> a3;
        std::vector<const double *> a1;
        std::vector<double> s;
    };
    std::vector<Bound> b(g->stages.size());
    for (size_t st = 0; st < g->stages.size(); st++) {
        const Plan &p = *g->stages[st];
        b[st].a3.assign(p.n3(), nullptr);
        b[st].a1.assign(p.n1(), nullptr);
        b[st].s.assign(p.ns(), 0.0);
        for (size_t q = 0; q < p.st.formals.size(); q++) {
            const Formal &f = p.st.formals[q];
            const ProgramArg &a = g->ir.args[g->ir.map[st][q]];
            if (f.kind == ArgKind::Array3D) b[st].a3[f.kind_index] = a3[a.kind_index];
            else if (f.kind == ArgKind::Array1D) b[st].a1[f.kind_index] = a1[a.kind_index];
            else b[st].s[f.kind_index] = s[a.kind_index];
        }
    }
    for (size_t st = 0; st < g->stages.size(); st++)
        plan_validate(g->stages[st].get(), b[st].a3.data(), int(b[st].a3.size()), b[st].a1.data(),
                      int(b[st].a1.size()), b[st].s.data(), int(b[st].s.size()), batch);
    for (size_t st = 0; st < g->stages.size(); st++)
        apply(g->stages[st].get(), b[st].a3.data(), int(b[st].a3.size()), b[st].a1.data(), int(b[st].a1.size()),
              b[st].s.data(), int(b[st].s.size()), batch, stream);
}

// Section VI-B: time every fusion-forest candidate of the program on the
// caller's arrays and report the fastest (the paper's tuning over fission
// versions).  Every candidate keeps the program's arguments.
void program_forest_tune(const std::string &text, const int64_t dims[3], const sdag_plan_opts &o, double *const *a3,
                         int n3, const double *const *a1, int n1, const double *s, int ns, cudaStream_t stream,
                         int max_candidates, double *ms, int *n_candidates, int *best) {
    const auto cands = forest_partitions(text, max_candidates);
    *n_candidates = int(cands.size());
    *best = -1;
    double best_ms = 0.0;
    struct Events {  // released on every path (a candidate's plan or launch may throw)
        cudaEvent_t e[2] = {nullptr, nullptr};
        ~Events() {
            for (cudaEvent_t x : e)
                if (x) cudaEventDestroy(x);
        }
    } ev;
    check_cuda(cudaEventCreate(&ev.e[0]), "cudaEventCreate");
    check_cuda(cudaEventCreate(&ev.e[1]), "cudaEventCreate");
    cudaEvent_t e0 = ev.e[0], e1 = ev.e[1];
    for (size_t c = 0; c < cands.size(); c++) {
        std::unique_ptr<Program> g(program_create(fuse_groups(text, cands[c]), dims, o));
        std::vector<float> t;
        for (int it = 0; it < 7; it++) {
            check_cuda(cudaEventRecord(e0, stream), "cudaEventRecord");
            program_apply(g.get(), a3, n3, a1, n1, s, ns, 1, stream);
            check_cuda(cudaEventRecord(e1, stream), "cudaEventRecord");
            check_cuda(cudaEventSynchronize(e1), "cudaEventSynchronize");
            float x = 0.f;
            check_cuda(cudaEventElapsedTime(&x, e0, e1), "cudaEventElapsedTime");
            if (it >= 2) t.push_back(x);
        }
        std::sort(t.begin(), t.end());
        const double med = t[t.size() / 2];
        if (ms) ms[c] = med;
        if (*best < 0 || med < best_ms) {
            *best = int(c);
            best_ms = med;
        }
    }
}

}  // namespace sdag
