// runtime.cpp -- the Paraprox runtime loop.
//
// PAPER.md §2: "the runtime system ... checks the output quality
// periodically ... If the quality drops below the TOQ, it uses a less
// aggressive approximation"; §5: checking every 40-50 invocations
// keeps the overhead under 5 % (SAGE).  The paper leaves the rest to Green /
// SAGE; the readings below are DESIGN.md R1-R4.
//
//  R1 train: the TOQ tuner (candidates in cost order, O7) on the
//     training frames; the first candidate with quality >= TOQ is rung 0.
//  R2 ladder: after it, the later candidates whose training quality is higher
//     than every rung before them (strictly less aggressive on the training
//     set), then EXACT.
//  R3 check: every check_every-th invocation (the 1st, then every
//     check_every-th after it) additionally runs the exact stencil on the same
//     input and the quality kernel on (exact, output) -- all on the caller's
//     stream, partials copied to pinned host memory with an event; the hot
//     path never waits for it.
//  R4 back-off: a check that finished (event complete at the next invocation,
//     or at paraprox_runtime_sync) with quality < TOQ moves one rung down the
//     ladder.  Exact never moves.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <mutex>
#include <new>
#include <vector>

#include "internal.h"

struct paraprox_runtime_s {
    paraprox_filter f = nullptr;
    double toq = 0.9;
    paraprox_metric m = PARAPROX_MRE;
    int check_every = 0;
    std::vector<ppx::Candidate> cands;
    std::vector<double> train_q;
    std::vector<int> ladder;  // candidate indices, -1 = exact (always last)
    int rung = 0;
    long long invocations = 0, checks = 0, backoffs = 0;
    double last_q = 0.0;
    bool trained = false;
    bool profiled = false;       // R1': pick the fastest passing candidate by measurement
    std::vector<double> time_ms;  // per candidate (profiled mode; NaN = not measured), then exact

    // check state
    float* d_exact = nullptr;
    size_t exact_cap = 0;
    double* d_part = nullptr;
    double* h_part = nullptr;
    cudaEvent_t ev = nullptr;
    bool pending = false;
    int dev = -1;
    std::mutex mu;
};

namespace ppx {

static void rt_release(paraprox_runtime rt) {
    if (rt->d_exact) cudaFree(rt->d_exact);
    if (rt->d_part) cudaFree(rt->d_part);
    if (rt->h_part) cudaFreeHost(rt->h_part);
    if (rt->ev) cudaEventDestroy(rt->ev);
    rt->d_exact = nullptr;
    rt->d_part = nullptr;
    rt->h_part = nullptr;
    rt->ev = nullptr;
    rt->exact_cap = 0;
}

// apply a finished check (R4); caller holds the lock
static void rt_apply(paraprox_runtime rt) {
    rt->pending = false;
    rt->last_q = quality_of(rt->h_part, rt->m);
    if (rt->last_q < rt->toq && rt->rung + 1 < (int)rt->ladder.size()) {
        ++rt->rung;
        ++rt->backoffs;
    }
}

static void rt_current(paraprox_runtime rt, paraprox_scheme* sc, int* reach) {
    const int k = rt->ladder[rt->rung];
    if (k < 0) {
        *sc = PARAPROX_EXACT;
        *reach = 0;
    } else {
        *sc = rt->cands[k].scheme;
        *reach = rt->cands[k].reach;
    }
}

}  // namespace ppx

using namespace ppx;

extern "C" {

paraprox_status paraprox_runtime_create(paraprox_filter f, double toq, paraprox_metric m, int check_every,
                                        paraprox_runtime* out) {
    if (!f || !out) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    paraprox_status st = check_toq(toq, m);
    if (st != PARAPROX_OK) return st;
    if (check_every < 0) return fail(PARAPROX_ERR_INVALID_ARG, "check_every < 0");
    paraprox_runtime rt = new (std::nothrow) paraprox_runtime_s;
    if (!rt) return fail(PARAPROX_ERR_ALLOC, "runtime allocation");
    rt->f = f;
    rt->toq = toq;
    rt->m = m;
    rt->check_every = check_every;
    *out = rt;
    return PARAPROX_OK;
}

void paraprox_runtime_destroy(paraprox_runtime rt) {
    if (!rt) return;
    if (rt->pending && rt->ev) cudaEventSynchronize(rt->ev);
    rt_release(rt);
    delete rt;
}

paraprox_status paraprox_runtime_train(paraprox_runtime rt, const float* d_train, const paraprox_image* img,
                                       paraprox_stream s) {
    if (!rt) return fail(PARAPROX_ERR_INVALID_ARG, "runtime is NULL");
    std::lock_guard<std::mutex> lk(rt->mu);
    if (rt->pending && rt->ev) cudaEventSynchronize(rt->ev);
    rt->pending = false;
    std::vector<Candidate> c = candidates(rt->f);
    std::vector<double> parts(3 * c.size() + 3);
    paraprox_status st = tune_partials_impl(rt->f, d_train, img, rt->m, c, parts.data(), s);
    if (st != PARAPROX_OK) return st;
    rt->cands = c;
    rt->train_q.assign(c.size(), 0.0);
    for (size_t k = 0; k < c.size(); ++k) rt->train_q[k] = quality_of(parts.data() + 3 * k, rt->m);
    // R1 / R2
    rt->ladder.clear();
    rt->time_ms.assign(c.size() + 1, NAN);
    int first = -1;
    if (!rt->profiled) {
        for (size_t k = 0; k < c.size(); ++k)
            if (rt->train_q[k] >= rt->toq) {
                first = (int)k;
                break;
            }
        if (first >= 0) {
            rt->ladder.push_back(first);
            double best = rt->train_q[first];
            for (size_t k = first + 1; k < c.size(); ++k)
                if (rt->train_q[k] > best) {
                    rt->ladder.push_back((int)k);
                    best = rt->train_q[k];
                }
        }
    } else {
        // R1' ("profiles the kernels and picks ... the best
        // performance"): every passing candidate and the exact stencil are
        // timed on the training frames (CUDA events, best of 3 after a warm-up
        // launch); rung 0 is the fastest passing one, the ladder continues
        // with the passing candidates of strictly higher training quality in
        // increasing quality, then EXACT
        cudaStream_t cs = (cudaStream_t)s;
        // timing output with the training image's layout (run_stencil shares it)
        const long long fs = img->n > 1 ? img->frame_stride : (long long)img->h * img->pitch;
        const long long need = (long long)(img->n - 1) * fs + (long long)(img->h - 1) * img->pitch + img->w;
        // scratch and events released on every return path
        struct Guard {
            void* tmp = nullptr;
            cudaStream_t cs = nullptr;
            cudaEvent_t e0 = nullptr, e1 = nullptr;
            ~Guard() {
                if (e0) cudaEventDestroy(e0);
                if (e1) cudaEventDestroy(e1);
                if (tmp) cudaFreeAsync(tmp, cs);
            }
        } g;
        g.cs = cs;
        PPX_CUDA(scratch_alloc(&g.tmp, sizeof(float) * need, cs));
        void* tmp = g.tmp;
        PPX_CUDA(cudaEventCreate(&g.e0));
        PPX_CUDA(cudaEventCreate(&g.e1));
        cudaEvent_t e0 = g.e0, e1 = g.e1;
        auto time_it = [&](int dy, int dx, double* ms) -> paraprox_status {
            float best = INFINITY;
            for (int rep = 0; rep < 4; ++rep) {
                PPX_CUDA(cudaEventRecord(e0, cs));
                paraprox_status st2 = run_stencil(rt->f, dy, dx, d_train, (float*)tmp, img, s);
                if (st2 != PARAPROX_OK) return st2;
                PPX_CUDA(cudaEventRecord(e1, cs));
                PPX_CUDA(cudaEventSynchronize(e1));
                float t = 0.f;
                PPX_CUDA(cudaEventElapsedTime(&t, e0, e1));
                if (rep > 0 && t < best) best = t;
            }
            *ms = best;
            return PARAPROX_OK;
        };
        paraprox_status st2 = PARAPROX_OK;
        double best_ms = INFINITY;
        for (size_t k = 0; k < c.size() && st2 == PARAPROX_OK; ++k) {
            if (rt->train_q[k] < rt->toq) continue;
            st2 = time_it(c[k].dy, c[k].dx, &rt->time_ms[k]);
            if (st2 == PARAPROX_OK && rt->time_ms[k] < best_ms) {
                best_ms = rt->time_ms[k];
                first = (int)k;
            }
        }
        if (st2 == PARAPROX_OK) st2 = time_it(0, 0, &rt->time_ms[c.size()]);
        if (st2 != PARAPROX_OK) return st2;
        if (first >= 0) {
            std::vector<int> up;
            for (size_t k = 0; k < c.size(); ++k)
                if ((int)k != first && rt->train_q[k] >= rt->toq && rt->train_q[k] > rt->train_q[first])
                    up.push_back((int)k);
            std::stable_sort(up.begin(), up.end(), [&](int a, int b) { return rt->train_q[a] < rt->train_q[b]; });
            rt->ladder.push_back(first);
            double best = rt->train_q[first];
            for (int k : up)
                if (rt->train_q[k] > best) {
                    rt->ladder.push_back(k);
                    best = rt->train_q[k];
                }
        }
    }
    rt->ladder.push_back(-1);
    rt->rung = 0;
    rt->invocations = rt->checks = rt->backoffs = 0;
    rt->last_q = first >= 0 ? rt->train_q[first] : (rt->m == PARAPROX_PSNR ? INFINITY : 1.0);
    rt->trained = true;
    return PARAPROX_OK;
}

paraprox_status paraprox_runtime_run(paraprox_runtime rt, const float* d_in, float* d_out, const paraprox_image* img,
                                     paraprox_stream s) {
    if (!rt) return fail(PARAPROX_ERR_INVALID_ARG, "runtime is NULL");
    std::lock_guard<std::mutex> lk(rt->mu);
    if (!rt->trained) return fail(PARAPROX_ERR_INVALID_ARG, "runtime not trained");
    if (rt->pending) {  // R4 without blocking: only a finished check is applied
        const cudaError_t q = cudaEventQuery(rt->ev);
        if (q == cudaSuccess) rt_apply(rt);
        else if (q != cudaErrorNotReady) return cuda_fail(q, "check event");
    }
    paraprox_scheme sc;
    int reach;
    rt_current(rt, &sc, &reach);
    int dy, dx;
    scheme_reaches(sc, reach, &dy, &dx);
    paraprox_status st = run_stencil(rt->f, dy, dx, d_in, d_out, img, s);
    if (st != PARAPROX_OK) return st;
    const bool check = rt->check_every > 0 && (rt->invocations % rt->check_every) == 0 && !rt->pending &&
                       sc != PARAPROX_EXACT;
    ++rt->invocations;
    if (!check) return PARAPROX_OK;
    // R3: exact on the same input into a buffer with the output's layout, then
    // the quality partials, copied to pinned host memory behind an event
    cudaStream_t cs = (cudaStream_t)s;
    int dev = 0;
    PPX_CUDA(cudaGetDevice(&dev));
    const long long ofs0 = img->n > 1 ? img->frame_stride : (long long)img->h * img->pitch;
    if (fused_quality_enabled()) {
        // fused check: the exact stencil of the same input is compared with
        // d_out in its epilogue and never stored
        if (rt->dev != dev) {
            if (rt->pending && rt->ev) cudaEventSynchronize(rt->ev);
            rt_release(rt);
            rt->dev = dev;
        }
        if (!rt->d_part) PPX_CUDA(cudaMalloc(&rt->d_part, 3 * sizeof(double)));
        if (!rt->h_part) PPX_CUDA(cudaMallocHost(&rt->h_part, 3 * sizeof(double)));
        if (!rt->ev) PPX_CUDA(cudaEventCreateWithFlags(&rt->ev, cudaEventDisableTiming));
        void* scratch = nullptr;
        PPX_CUDA(scratch_alloc(&scratch, sizeof(double) * quality_scratch_doubles((long long)img->n * img->h * img->w), cs));
        bool fused = false;
        cudaError_t e = launch_stencil_quality(get_plan(rt->f, 0, 0), d_in, view_of(img), d_out, img->pitch, ofs0,
                                               rt->m, false, rt->d_part, (double*)scratch, cs, &fused);
        if (fused || e != cudaSuccess) {
            cudaFreeAsync(scratch, cs);
            if (e != cudaSuccess) return cuda_fail(e, "fused check launch");
            PPX_CUDA(cudaMemcpyAsync(rt->h_part, rt->d_part, 3 * sizeof(double), cudaMemcpyDeviceToHost, cs));
            PPX_CUDA(cudaEventRecord(rt->ev, cs));
            rt->pending = true;
            ++rt->checks;
            return PARAPROX_OK;
        }
        cudaFreeAsync(scratch, cs);
    }
    if (rt->dev != dev) {
        if (rt->pending && rt->ev) cudaEventSynchronize(rt->ev);
        rt_release(rt);
        rt->dev = dev;
    }
    const long long ofs = img->n > 1 ? img->frame_stride : (long long)img->h * img->pitch;
    const size_t need = (size_t)((img->n - 1) * ofs + (long long)(img->h - 1) * img->pitch + img->w);
    if (need > rt->exact_cap) {
        if (rt->d_exact) {
            PPX_CUDA(cudaStreamSynchronize(cs));
            cudaFree(rt->d_exact);
            rt->d_exact = nullptr;
        }
        PPX_CUDA(cudaMalloc(&rt->d_exact, need * sizeof(float)));
        rt->exact_cap = need;
    }
    if (!rt->d_part) PPX_CUDA(cudaMalloc(&rt->d_part, 3 * sizeof(double)));
    if (!rt->h_part) PPX_CUDA(cudaMallocHost(&rt->h_part, 3 * sizeof(double)));
    if (!rt->ev) PPX_CUDA(cudaEventCreateWithFlags(&rt->ev, cudaEventDisableTiming));
    const View v = view_of(img);
    cudaError_t e = launch_stencil(get_plan(rt->f, 0, 0), d_in, v, rt->d_exact, img->pitch, ofs, cs);
    if (e != cudaSuccess) return cuda_fail(e, "check exact launch");
    View vq = v;  // the outputs' layout: rows 0..h-1 only
    vq.fstride = ofs;
    vq.lo = 0;
    vq.hi = img->h - 1;
    void* scratch = nullptr;
    PPX_CUDA(scratch_alloc(&scratch, sizeof(double) * quality_scratch_doubles((long long)img->n * img->h * img->w), cs));
    e = launch_quality(rt->d_exact, d_out, vq, rt->m, rt->d_part, (double*)scratch, cs);
    cudaFreeAsync(scratch, cs);
    if (e != cudaSuccess) return cuda_fail(e, "check quality launch");
    PPX_CUDA(cudaMemcpyAsync(rt->h_part, rt->d_part, 3 * sizeof(double), cudaMemcpyDeviceToHost, cs));
    PPX_CUDA(cudaEventRecord(rt->ev, cs));
    rt->pending = true;
    ++rt->checks;
    return PARAPROX_OK;
}

paraprox_status paraprox_runtime_sync(paraprox_runtime rt) {
    if (!rt) return fail(PARAPROX_ERR_INVALID_ARG, "runtime is NULL");
    std::lock_guard<std::mutex> lk(rt->mu);
    if (rt->pending) {
        PPX_CUDA(cudaEventSynchronize(rt->ev));
        rt_apply(rt);
    }
    return PARAPROX_OK;
}

paraprox_status paraprox_runtime_state(paraprox_runtime rt, paraprox_scheme* scheme, int* reach,
                                       long long* invocations, long long* checks, long long* backoffs,
                                       double* last_quality) {
    if (!rt) return fail(PARAPROX_ERR_INVALID_ARG, "runtime is NULL");
    std::lock_guard<std::mutex> lk(rt->mu);
    if (!rt->trained) return fail(PARAPROX_ERR_INVALID_ARG, "runtime not trained");
    paraprox_scheme sc;
    int r;
    rt_current(rt, &sc, &r);
    if (scheme) *scheme = sc;
    if (reach) *reach = r;
    if (invocations) *invocations = rt->invocations;
    if (checks) *checks = rt->checks;
    if (backoffs) *backoffs = rt->backoffs;
    if (last_quality) *last_quality = rt->last_q;
    return PARAPROX_OK;
}

paraprox_status paraprox_runtime_set_profiled(paraprox_runtime rt, int enable) {
    if (!rt) return fail(PARAPROX_ERR_INVALID_ARG, "runtime is NULL");
    std::lock_guard<std::mutex> lk(rt->mu);
    rt->profiled = enable != 0;
    return PARAPROX_OK;
}

paraprox_status paraprox_runtime_timings(paraprox_runtime rt, int cap, int* n, double* ms) {
    if (!rt || !n) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    std::lock_guard<std::mutex> lk(rt->mu);
    if (!rt->trained) return fail(PARAPROX_ERR_INVALID_ARG, "runtime not trained");
    *n = (int)rt->time_ms.size();
    for (int i = 0; i < *n && i < cap; ++i)
        if (ms) ms[i] = rt->time_ms[i];
    return PARAPROX_OK;
}

paraprox_status paraprox_runtime_ladder(paraprox_runtime rt, int cap, int* n, paraprox_scheme* schemes,
                                        int* reaches, double* train_quality) {
    if (!rt || !n) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (cap < 0) return fail(PARAPROX_ERR_INVALID_ARG, "cap < 0");
    std::lock_guard<std::mutex> lk(rt->mu);
    if (!rt->trained) return fail(PARAPROX_ERR_INVALID_ARG, "runtime not trained");
    *n = (int)rt->ladder.size();
    for (int i = 0; i < *n && i < cap; ++i) {
        const int k = rt->ladder[i];
        if (schemes) schemes[i] = k < 0 ? PARAPROX_EXACT : rt->cands[k].scheme;
        if (reaches) reaches[i] = k < 0 ? 0 : rt->cands[k].reach;
        if (train_quality) train_quality[i] = k < 0 ? (rt->m == PARAPROX_PSNR ? INFINITY : 1.0) : rt->train_q[k];
    }
    return PARAPROX_OK;
}

}  // extern "C"
