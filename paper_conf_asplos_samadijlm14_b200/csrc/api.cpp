// api.cpp -- the extern "C" entry points of libparaprox (include/paraprox.h):
// argument validation, plan lookup, stream-ordered scratch, the TOQ tuner and
// the host-buffer end-to-end path.  All arithmetic runs in the kernels.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <new>
#include <mutex>
#include <string>

#include "internal.h"

namespace ppx {

std::atomic<unsigned long long> g_launches{0};
thread_local const char* t_last_kernel = "none";
static thread_local std::string t_err;

void count_launch(const char* name) {
    g_launches.fetch_add(1, std::memory_order_relaxed);
    t_last_kernel = name;
}

paraprox_status fail(paraprox_status st, const std::string& msg) {
    t_err = msg;
    return st;
}

paraprox_status cuda_fail(cudaError_t e, const char* where) {
    t_err = std::string(where) + ": " + cudaGetErrorString(e);
    return e == cudaErrorMemoryAllocation ? PARAPROX_ERR_ALLOC : PARAPROX_ERR_CUDA;
}



static bool odd_k(int k) { return k >= 1 && (k & 1) == 1; }

paraprox_status check_image(const paraprox_image* img, bool allow_halo) {
    if (!img) return fail(PARAPROX_ERR_INVALID_ARG, "img is NULL");
    if (img->n < 1 || img->h < 1 || img->w < 1) return fail(PARAPROX_ERR_INVALID_ARG, "n, h, w must be >= 1");
    if (img->pitch < img->w) return fail(PARAPROX_ERR_INVALID_ARG, "pitch < w");
    if (img->halo_top < 0 || img->halo_bottom < 0) return fail(PARAPROX_ERR_INVALID_ARG, "negative halo");
    if (!allow_halo && (img->halo_top || img->halo_bottom))
        return fail(PARAPROX_ERR_INVALID_ARG, "halos not allowed here");
    const long long rows = (long long)img->h + img->halo_top + img->halo_bottom;
    if (img->n > 1 && img->frame_stride < rows * img->pitch)
        return fail(PARAPROX_ERR_INVALID_ARG, "frame_stride < (h + halos) * pitch");
    return PARAPROX_OK;
}

View view_of(const paraprox_image* img) {
    View v;
    v.n = img->n;
    v.h = img->h;
    v.w = img->w;
    v.pitch = img->pitch;
    v.fstride = img->n > 1 ? img->frame_stride : (long long)(img->h + img->halo_bottom) * img->pitch;
    v.lo = -img->halo_top;
    v.hi = img->h - 1 + img->halo_bottom;
    return v;
}

// byte ranges touched: inputs (with halos) and outputs must not overlap
bool overlaps(const float* in, const float* out, const paraprox_image* img) {
    const long long fs = img->n > 1 ? img->frame_stride : 0;
    const char* i0 = (const char*)(in - (long long)img->halo_top * img->pitch);
    const char* i1 = (const char*)(in + (img->n - 1) * fs + (long long)(img->h - 1 + img->halo_bottom) * img->pitch + img->w);
    const char* o0 = (const char*)out;
    const char* o1 = (const char*)(out + (img->n - 1) * fs + (long long)(img->h - 1) * img->pitch + img->w);
    return i0 < o1 && o0 < i1;
}

// skip = false: (a, b) are reaches (dy, dx); skip = true: skipping rates (sy, sx)
static paraprox_status run_plan(paraprox_filter f, bool skip, int a, int b, const float* in, float* out,
                                const paraprox_image* img, paraprox_stream s) {
    if (!f) return fail(PARAPROX_ERR_INVALID_ARG, "filter is NULL");
    if (!in || !out) return fail(PARAPROX_ERR_INVALID_ARG, "NULL buffer");
    if (!skip && (a < 0 || b < 0)) return fail(PARAPROX_ERR_INVALID_ARG, "reach < 0");
    if (skip && (a < 1 || b < 1)) return fail(PARAPROX_ERR_INVALID_ARG, "skipping rate < 1");
    paraprox_status st = check_image(img, true);
    if (st != PARAPROX_OK) return st;
    if (overlaps(in, out, img)) return fail(PARAPROX_ERR_INVALID_ARG, "d_out overlaps d_in");
    const Plan& p = skip ? get_plan_skip(f, a, b) : get_plan(f, a, b);
    const View v = view_of(img);
    const long long ofs = img->n > 1 ? img->frame_stride : (long long)img->h * img->pitch;
    cudaError_t e = launch_stencil(p, in, v, out, img->pitch, ofs, (cudaStream_t)s);
    if (e != cudaSuccess) return cuda_fail(e, "stencil launch");
    return PARAPROX_OK;
}

paraprox_status run_stencil(paraprox_filter f, int dy, int dx, const float* in, float* out,
                            const paraprox_image* img, paraprox_stream s) {
    return run_plan(f, false, dy, dx, in, out, img, s);
}

// any scheme, stencil (reach) or reduction (skipping rate)
static paraprox_status run_scheme(paraprox_filter f, paraprox_scheme scheme, int reach, const float* in, float* out,
                                  const paraprox_image* img, paraprox_stream s) {
    if (scheme < PARAPROX_EXACT || scheme > PARAPROX_SKIP_BOTH) return fail(PARAPROX_ERR_INVALID_ARG, "unknown scheme");
    if (is_skip_scheme(scheme)) {
        if (reach < 1) return fail(PARAPROX_ERR_INVALID_ARG, "skipping rate < 1");
        int sy, sx;
        scheme_skips(scheme, reach, &sy, &sx);
        return run_plan(f, true, sy, sx, in, out, img, s);
    }
    if (reach < 0) return fail(PARAPROX_ERR_INVALID_ARG, "reach < 0");
    int dy, dx;
    scheme_reaches(scheme, reach, &dy, &dx);
    return run_plan(f, false, dy, dx, in, out, img, s);
}

static const Plan& cand_plan(paraprox_filter f, const Candidate& c) {
    return is_skip_scheme(c.scheme) ? get_plan_skip(f, c.dy, c.dx) : get_plan(f, c.dy, c.dx);
}

bool fused_quality_enabled() { return knobs().fused_quality; }

constexpr int kMaxLatticeReach = 1 << 20;

static paraprox_status run_lattice(paraprox_filter f, int dy, int dx, const float* in, float* out,
                                   const paraprox_image* img, paraprox_stream s) {
    if (!f) return fail(PARAPROX_ERR_INVALID_ARG, "filter is NULL");
    if (!in || !out) return fail(PARAPROX_ERR_INVALID_ARG, "NULL buffer");
    if (dy < 0 || dx < 0) return fail(PARAPROX_ERR_INVALID_ARG, "reach < 0");
    if (dy > kMaxLatticeReach || dx > kMaxLatticeReach) return fail(PARAPROX_ERR_INVALID_ARG, "reach too large");
    paraprox_status st = check_image(img, false);
    if (st != PARAPROX_OK) return st;
    if (overlaps(in, out, img)) return fail(PARAPROX_ERR_INVALID_ARG, "d_out overlaps d_in");
    const View v = view_of(img);
    const long long ofs = img->n > 1 ? img->frame_stride : (long long)img->h * img->pitch;
    cudaError_t e = (dy == 0 && dx == 0)
                        ? launch_stencil(get_plan(f, 0, 0), in, v, out, img->pitch, ofs, (cudaStream_t)s)
                        : launch_lattice(*f, in, v, out, img->pitch, ofs, dy, dx, (cudaStream_t)s);
    if (e != cudaSuccess) return cuda_fail(e, "lattice launch");
    return PARAPROX_OK;
}

double quality_of(const double* p3, paraprox_metric m) {
    if (m == PARAPROX_MRE) return 1.0 - p3[0] / p3[1];
    if (m == PARAPROX_L2) {
        if (p3[1] == 0.0) return p3[0] == 0.0 ? 1.0 : -INFINITY;
        return 1.0 - std::sqrt(p3[0] / p3[1]);
    }
    const double mse = p3[0] / p3[1];
    return mse == 0.0 ? INFINITY : 10.0 * std::log10(255.0 * 255.0 / mse);
}

bool metric_ok(paraprox_metric m) { return m == PARAPROX_MRE || m == PARAPROX_L2 || m == PARAPROX_PSNR; }

// Stream-ordered scratch comes from a library-owned memory pool per device
// whose release threshold keeps freed blocks mapped, so repeated calls (the
// tuner, run_host) do not remap device memory every time.
cudaError_t scratch_alloc(void** p, size_t bytes, cudaStream_t s) {
    static std::mutex mu;
    static cudaMemPool_t pools[64] = {};
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    if (dev >= 64) return cudaMallocAsync(p, bytes, s);
    {
        std::lock_guard<std::mutex> lk(mu);
        if (!pools[dev]) {
            cudaMemPoolProps props = {};
            props.allocType = cudaMemAllocationTypePinned;
            props.location.type = cudaMemLocationTypeDevice;
            props.location.id = dev;
            e = cudaMemPoolCreate(&pools[dev], &props);
            if (e != cudaSuccess) return e;
            uint64_t keep = ~0ull;
            cudaMemPoolSetAttribute(pools[dev], cudaMemPoolAttrReleaseThreshold, &keep);
        }
    }
    return cudaMallocFromPoolAsync(p, bytes, pools[dev], s);
}

struct DevBuf {
    void* p = nullptr;
    cudaStream_t s = nullptr;
    ~DevBuf() {
        if (p) cudaFreeAsync(p, s);
    }
};

static paraprox_status quality_partials_impl(const float* e, const float* a, const paraprox_image* img,
                                             paraprox_metric m, double* h3, paraprox_stream s) {
    if (!e || !a || !h3) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (!metric_ok(m)) return fail(PARAPROX_ERR_INVALID_ARG, "unknown metric");
    paraprox_status st = check_image(img, false);
    if (st != PARAPROX_OK) return st;
    cudaStream_t cs = (cudaStream_t)s;
    DevBuf buf;
    buf.s = cs;
    const size_t qsd = quality_scratch_doubles((long long)img->n * img->h * img->w);
    PPX_CUDA(scratch_alloc(&buf.p, sizeof(double) * (qsd + 3), cs));
    double* d = (double*)buf.p;
    cudaError_t err = launch_quality(e, a, view_of(img), m, d + qsd, d, cs);
    if (err != cudaSuccess) return cuda_fail(err, "quality launch");
    PPX_CUDA(cudaMemcpyAsync(h3, d + qsd, 3 * sizeof(double), cudaMemcpyDeviceToHost, cs));
    PPX_CUDA(cudaStreamSynchronize(cs));
    return PARAPROX_OK;
}

// all candidates' partials into h_partials[3 * n]
paraprox_status tune_partials_impl(paraprox_filter f, const float* d_train, const paraprox_image* img,
                                          paraprox_metric m, const std::vector<Candidate>& cands,
                                          double* h_partials, paraprox_stream s, double stop_toq) {
    if (!f || !d_train || (!h_partials && !cands.empty())) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (!metric_ok(m)) return fail(PARAPROX_ERR_INVALID_ARG, "unknown metric");
    paraprox_status st = check_image(img, true);
    if (st != PARAPROX_OK) return st;
    if (cands.empty()) return PARAPROX_OK;
    cudaStream_t cs = (cudaStream_t)s;
    const long long plane = (long long)img->h * img->w;
    const long long count = plane * img->n;
    const size_t nc = cands.size();
    DevBuf buf;
    buf.s = cs;
    const size_t qsd = quality_scratch_doubles(count);
    const size_t bytes = sizeof(float) * 2 * count + sizeof(double) * (qsd + 3 * nc) + 256;
    PPX_CUDA(scratch_alloc(&buf.p, bytes, cs));
    float* E = (float*)buf.p;
    float* A = E + count;
    double* scratch = (double*)(((uintptr_t)(A + count) + 255) & ~(uintptr_t)255);
    double* parts = scratch + qsd;
    const View vin = view_of(img);
    View vq;  // compact layout of the scratch outputs
    vq.n = img->n;
    vq.h = img->h;
    vq.w = img->w;
    vq.pitch = img->w;
    vq.fstride = plane;
    vq.lo = 0;
    vq.hi = img->h - 1;
    cudaError_t e = launch_stencil(get_plan(f, 0, 0), d_train, vin, E, img->w, plane, cs);
    if (e != cudaSuccess) return cuda_fail(e, "exact launch");
    for (size_t k = 0; k < nc; ++k) {
        // fused: the candidate's output is compared with E in the stencil's
        // epilogue and never stored (8 B/px instead of 16)
        bool fused = false;
        if (fused_quality_enabled()) {
            e = launch_stencil_quality(cand_plan(f, cands[k]), d_train, vin, E, img->w, plane, m, true,
                                       parts + 3 * k, scratch, cs, &fused);
            if (e != cudaSuccess) return cuda_fail(e, "fused candidate launch");
        }
        if (!fused) {
            e = launch_stencil(cand_plan(f, cands[k]), d_train, vin, A, img->w, plane, cs);
            if (e != cudaSuccess) return cuda_fail(e, "candidate launch");
            e = launch_quality(E, A, vq, m, parts + 3 * k, scratch, cs);
            if (e != cudaSuccess) return cuda_fail(e, "quality launch");
        }
        if (!std::isnan(stop_toq)) {
            // early exit (paraprox_tune): the decision is the first candidate
            // in cost order with Q >= TOQ, so nothing after it is needed; the
            // partials of candidates 0..k are the same bits as in a full scan
            PPX_CUDA(cudaMemcpyAsync(h_partials + 3 * k, parts + 3 * k, sizeof(double) * 3, cudaMemcpyDeviceToHost, cs));
            PPX_CUDA(cudaStreamSynchronize(cs));
            if (quality_of(h_partials + 3 * k, m) >= stop_toq) {
                for (size_t j = k + 1; j < nc; ++j) h_partials[3 * j] = h_partials[3 * j + 1] = h_partials[3 * j + 2] = NAN;
                return PARAPROX_OK;
            }
        }
    }
    if (!std::isnan(stop_toq)) return PARAPROX_OK;  // every candidate copied above
    PPX_CUDA(cudaMemcpyAsync(h_partials, parts, sizeof(double) * 3 * nc, cudaMemcpyDeviceToHost, cs));
    PPX_CUDA(cudaStreamSynchronize(cs));
    return PARAPROX_OK;
}

// the lattice tuner's candidates: row lattice reach 4, 3, 2, 1 (fewest HBM
// bytes first, 4/(2d+1) + 4 B per pixel)
constexpr int kLatticeCands = 4;

static paraprox_status lattice_partials_impl(paraprox_filter f, const float* d_train, const paraprox_image* img,
                                             paraprox_metric m, double* h_partials, paraprox_stream s) {
    if (!f || !d_train || !h_partials) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (!metric_ok(m)) return fail(PARAPROX_ERR_INVALID_ARG, "unknown metric");
    paraprox_status st = check_image(img, false);
    if (st != PARAPROX_OK) return st;
    cudaStream_t cs = (cudaStream_t)s;
    const long long plane = (long long)img->h * img->w;
    const long long count = plane * img->n;
    DevBuf buf;
    buf.s = cs;
    const size_t qsd = quality_scratch_doubles(count);
    const size_t bytes = sizeof(float) * 2 * count + sizeof(double) * (qsd + 3 * kLatticeCands) + 256;
    PPX_CUDA(scratch_alloc(&buf.p, bytes, cs));
    float* E = (float*)buf.p;
    float* A = E + count;
    double* scratch = (double*)(((uintptr_t)(A + count) + 255) & ~(uintptr_t)255);
    double* parts = scratch + qsd;
    const View vin = view_of(img);
    View vq;
    vq.n = img->n;
    vq.h = img->h;
    vq.w = img->w;
    vq.pitch = img->w;
    vq.fstride = plane;
    vq.lo = 0;
    vq.hi = img->h - 1;
    cudaError_t e = launch_stencil(get_plan(f, 0, 0), d_train, vin, E, img->w, plane, cs);
    if (e != cudaSuccess) return cuda_fail(e, "exact launch");
    for (int k = 0; k < kLatticeCands; ++k) {
        e = launch_lattice(*f, d_train, vin, A, img->w, plane, kLatticeCands - k, 0, cs);
        if (e != cudaSuccess) return cuda_fail(e, "lattice launch");
        e = launch_quality(E, A, vq, m, parts + 3 * k, scratch, cs);
        if (e != cudaSuccess) return cuda_fail(e, "quality launch");
    }
    PPX_CUDA(cudaMemcpyAsync(h_partials, parts, sizeof(double) * 3 * kLatticeCands, cudaMemcpyDeviceToHost, cs));
    PPX_CUDA(cudaStreamSynchronize(cs));
    return PARAPROX_OK;
}

static paraprox_status decide(const std::vector<Candidate>& cands, const double* parts, paraprox_metric m,
                              double toq, paraprox_scheme* sc, int* reach, double* q) {
    *sc = PARAPROX_EXACT;
    *reach = 0;
    *q = m == PARAPROX_PSNR ? INFINITY : 1.0;
    for (size_t k = 0; k < cands.size(); ++k) {
        const double qk = quality_of(parts + 3 * k, m);
        if (qk >= toq) {
            *sc = cands[k].scheme;
            *reach = cands[k].reach;
            *q = qk;
            return PARAPROX_OK;
        }
    }
    return PARAPROX_OK;
}

paraprox_status check_toq(double toq, paraprox_metric m) {
    if (!metric_ok(m)) return fail(PARAPROX_ERR_INVALID_ARG, "unknown metric");
    if (m != PARAPROX_PSNR && !(toq > 0.0 && toq <= 1.0)) return fail(PARAPROX_ERR_INVALID_ARG, "toq not in (0, 1]");
    if (std::isnan(toq)) return fail(PARAPROX_ERR_INVALID_ARG, "toq is NaN");
    return PARAPROX_OK;
}

}  // namespace ppx

using namespace ppx;

extern "C" {

paraprox_status paraprox_filter_create(int ky, int kx, const float* h_w, paraprox_filter* out) {
    if (!h_w || !out) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (!odd_k(ky) || !odd_k(kx)) return fail(PARAPROX_ERR_INVALID_ARG, "K must be odd and >= 1");
    if (ky > kMaxK || kx > kMaxK) return fail(PARAPROX_ERR_UNSUPPORTED, "K > 17");
    paraprox_filter f = new (std::nothrow) paraprox_filter_s;
    if (!f) return fail(PARAPROX_ERR_ALLOC, "filter allocation");
    f->ky = ky;
    f->kx = kx;
    f->separable = false;
    f->w.assign(h_w, h_w + (size_t)ky * kx);
    *out = f;
    return PARAPROX_OK;
}

paraprox_status paraprox_filter_create_separable(int ky, const float* h_wy, int kx, const float* h_wx,
                                                 paraprox_filter* out) {
    if (!h_wy || !h_wx || !out) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (!odd_k(ky) || !odd_k(kx)) return fail(PARAPROX_ERR_INVALID_ARG, "K must be odd and >= 1");
    if (ky > kMaxK || kx > kMaxK) return fail(PARAPROX_ERR_UNSUPPORTED, "K > 17");
    paraprox_filter f = new (std::nothrow) paraprox_filter_s;
    if (!f) return fail(PARAPROX_ERR_ALLOC, "filter allocation");
    f->ky = ky;
    f->kx = kx;
    f->separable = true;
    f->wy.assign(h_wy, h_wy + ky);
    f->wx.assign(h_wx, h_wx + kx);
    *out = f;
    return PARAPROX_OK;
}

void paraprox_filter_destroy(paraprox_filter f) { delete f; }

paraprox_status paraprox_filter_shape(paraprox_filter f, int* ky, int* kx, int* separable) {
    if (!f) return fail(PARAPROX_ERR_INVALID_ARG, "filter is NULL");
    if (ky) *ky = f->ky;
    if (kx) *kx = f->kx;
    if (separable) *separable = f->separable ? 1 : 0;
    return PARAPROX_OK;
}

paraprox_status paraprox_plan_info(paraprox_filter f, int reach_y, int reach_x, int* taps, int* halo_y,
                                   int* halo_x, int* h_map_y, int* h_map_x) {
    if (!f) return fail(PARAPROX_ERR_INVALID_ARG, "filter is NULL");
    if (reach_y < 0 || reach_x < 0) return fail(PARAPROX_ERR_INVALID_ARG, "reach < 0");
    const Plan& p = get_plan(f, reach_y, reach_x);
    if (taps) *taps = p.taps;
    if (halo_y) *halo_y = p.hy;
    if (halo_x) *halo_x = p.hx;
    if (h_map_y) std::copy(p.my, p.my + p.ky, h_map_y);
    if (h_map_x) std::copy(p.mx, p.mx + p.kx, h_map_x);
    return PARAPROX_OK;
}

paraprox_status paraprox_stencil_exact(paraprox_filter f, const float* d_in, float* d_out,
                                       const paraprox_image* img, paraprox_stream s) {
    return run_stencil(f, 0, 0, d_in, d_out, img, s);
}

paraprox_status paraprox_stencil_approx(paraprox_filter f, paraprox_scheme scheme, int reach, const float* d_in,
                                        float* d_out, const paraprox_image* img, paraprox_stream s) {
    return run_scheme(f, scheme, reach, d_in, d_out, img, s);
}

paraprox_status paraprox_stencil_skip_xy(paraprox_filter f, int skip_y, int skip_x, const float* d_in, float* d_out,
                                         const paraprox_image* img, paraprox_stream s) {
    return run_plan(f, true, skip_y, skip_x, d_in, d_out, img, s);
}

paraprox_status paraprox_stencil_approx_xy(paraprox_filter f, int reach_y, int reach_x, const float* d_in,
                                           float* d_out, const paraprox_image* img, paraprox_stream s) {
    return run_stencil(f, reach_y, reach_x, d_in, d_out, img, s);
}

paraprox_status paraprox_stencil_lattice(paraprox_filter f, paraprox_scheme scheme, int reach, const float* d_in,
                                         float* d_out, const paraprox_image* img, paraprox_stream s) {
    if (scheme < PARAPROX_EXACT || scheme > PARAPROX_CENTER) return fail(PARAPROX_ERR_INVALID_ARG, "unknown scheme");
    if (reach < 0) return fail(PARAPROX_ERR_INVALID_ARG, "reach < 0");
    int dy, dx;
    scheme_reaches(scheme, reach, &dy, &dx);
    return run_lattice(f, dy, dx, d_in, d_out, img, s);
}

paraprox_status paraprox_stencil_lattice_xy(paraprox_filter f, int reach_y, int reach_x, const float* d_in,
                                            float* d_out, const paraprox_image* img, paraprox_stream s) {
    return run_lattice(f, reach_y, reach_x, d_in, d_out, img, s);
}

paraprox_status paraprox_tune_lattice_partials(paraprox_filter f, const float* d_train, const paraprox_image* img,
                                               paraprox_metric m, double* h_partials12, paraprox_stream s) {
    return lattice_partials_impl(f, d_train, img, m, h_partials12, s);
}

paraprox_status paraprox_tune_lattice_decide(const double* h_partials12, paraprox_metric m, double toq,
                                             paraprox_scheme* out_scheme, int* out_reach, double* out_quality) {
    if (!h_partials12 || !out_scheme || !out_reach || !out_quality) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    paraprox_status st = check_toq(toq, m);
    if (st != PARAPROX_OK) return st;
    *out_scheme = PARAPROX_EXACT;
    *out_reach = 0;
    *out_quality = m == PARAPROX_PSNR ? INFINITY : 1.0;
    for (int k = 0; k < kLatticeCands; ++k) {
        const double q = quality_of(h_partials12 + 3 * k, m);
        if (q >= toq) {
            *out_scheme = PARAPROX_ROW;
            *out_reach = kLatticeCands - k;
            *out_quality = q;
            break;
        }
    }
    return PARAPROX_OK;
}

paraprox_status paraprox_tune_lattice(paraprox_filter f, const float* d_train, const paraprox_image* img, double toq,
                                      paraprox_metric m, paraprox_scheme* out_scheme, int* out_reach,
                                      double* out_quality, paraprox_stream s) {
    if (!out_scheme || !out_reach || !out_quality) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    paraprox_status st = check_toq(toq, m);
    if (st != PARAPROX_OK) return st;
    double parts[3 * kLatticeCands];
    st = lattice_partials_impl(f, d_train, img, m, parts, s);
    if (st != PARAPROX_OK) return st;
    return paraprox_tune_lattice_decide(parts, m, toq, out_scheme, out_reach, out_quality);
}

static bool hotspot_tb_enabled() { return knobs().hotspot_tb; }

paraprox_status paraprox_hotspot(const paraprox_hotspot_params* prm, paraprox_scheme scheme, int reach,
                                 const float* d_temp, const float* d_power, float* d_out, const paraprox_image* img,
                                 int iterations, paraprox_stream s) {
    if (!prm || !d_temp || !d_power || !d_out) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (scheme < PARAPROX_EXACT || scheme > PARAPROX_CENTER) return fail(PARAPROX_ERR_INVALID_ARG, "unknown scheme");
    if (reach < 0) return fail(PARAPROX_ERR_INVALID_ARG, "reach < 0");
    if (iterations < 1) return fail(PARAPROX_ERR_INVALID_ARG, "iterations < 1");
    paraprox_status st = check_image(img, iterations == 1);
    if (st != PARAPROX_OK) return st;
    if (overlaps(d_temp, d_out, img)) return fail(PARAPROX_ERR_INVALID_ARG, "d_out overlaps d_temp");
    paraprox_image pimg = *img;  // the power grid has the output's rows only
    pimg.halo_top = pimg.halo_bottom = 0;
    if (overlaps(d_power, d_out, &pimg)) return fail(PARAPROX_ERR_INVALID_ARG, "d_out overlaps d_power");
    // the step as a 3x3 filter on T plus an additive power term (reading S25):
    // T' = sum w T + c P + c gz Tamb, w = [[0, c gy, 0], [c gx, 1 - 2c gx - 2c gy - c gz, c gx], [0, c gy, 0]]
    const double c = prm->step_div_cap, gx = prm->rx_inv, gy = prm->ry_inv, gz = prm->rz_inv;
    paraprox_filter_s f;
    f.ky = f.kx = 3;
    f.separable = false;
    f.w = {0.f, (float)(c * gy), 0.f, (float)(c * gx), (float)(1.0 - 2.0 * c * gx - 2.0 * c * gy - c * gz),
           (float)(c * gx), 0.f, (float)(c * gy), 0.f};
    int dy, dx;
    scheme_reaches(scheme, reach, &dy, &dx);
    const Plan& p = get_plan(&f, dy, dx);
    cudaStream_t cs = (cudaStream_t)s;
    const View v0 = view_of(img);
    const long long ofs = img->n > 1 ? img->frame_stride : (long long)img->h * img->pitch;
    Addend add;
    add.p = d_power;
    add.pitch = img->pitch;
    add.fstride = ofs;
    add.alpha = (float)c;
    add.beta = (float)(c * gz * prm->t_amb);
    // ping-pong between d_out and one scratch image so that the last step
    // lands in d_out; d_temp is never written
    DevBuf buf;
    buf.s = cs;
    if (iterations > 1) {
        const size_t need = (size_t)((img->n - 1) * ofs + (long long)(img->h - 1) * img->pitch + img->w);
        PPX_CUDA(scratch_alloc(&buf.p, need * sizeof(float), cs));
    }
    View vn = v0;  // later steps read an image with the output's layout, no halos
    vn.fstride = ofs;
    vn.lo = 0;
    vn.hi = img->h - 1;
    const float* src = d_temp;
    if (p.hy == 0 && p.hx == 0) {
        // the centre scheme at full reach reads no neighbour: all the steps
        // fuse into one pass (k_pointwise), one HBM round trip for `iterations`
        add.steps = iterations;
        cudaError_t e = launch_stencil(p, src, v0, d_out, img->pitch, ofs, cs, &add);
        if (e != cudaSuccess) return cuda_fail(e, "hotspot fused steps");
        return PARAPROX_OK;
    }
    if (iterations > 1 && hotspot_tb_enabled()) {
        // temporal blocking (k_hotspot.cu): up to 8 steps per HBM pass; the
        // passes ping-pong so that the last lands in d_out
        const int passes = (iterations + kHotspotMaxSteps - 1) / kHotspotMaxSteps;
        for (int q = 0; q < passes; ++q) {
            const int steps = std::min(kHotspotMaxSteps, iterations - q * kHotspotMaxSteps);
            float* dst = ((passes - 1 - q) % 2 == 0) ? d_out : (float*)buf.p;
            cudaError_t e = launch_hotspot_tb(p, src, d_power, dst, vn, ofs, add.alpha, add.beta, steps, cs);
            if (e != cudaSuccess) return cuda_fail(e, "hotspot blocked steps");
            src = dst;
        }
        return PARAPROX_OK;
    }
    for (int it = 0; it < iterations; ++it) {
        float* dst = ((iterations - 1 - it) % 2 == 0) ? d_out : (float*)buf.p;
        cudaError_t e = launch_stencil(p, src, it == 0 ? v0 : vn, dst, img->pitch, ofs, cs, &add);
        if (e != cudaSuccess) return cuda_fail(e, "hotspot step");
        src = dst;
    }
    return PARAPROX_OK;
}

paraprox_status paraprox_stencil_peer(paraprox_filter f, paraprox_scheme scheme, int reach, const float* d_in,
                                      float* d_out, const paraprox_image* img, const float* d_top, int top_rows,
                                      const float* d_bot, int bot_rows, long long src_pitch, paraprox_stream s) {
    if (!f || !d_in || !d_out || !img) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (scheme < PARAPROX_EXACT || scheme > PARAPROX_CENTER) return fail(PARAPROX_ERR_INVALID_ARG, "unknown scheme");
    if (reach < 0 || top_rows < 0 || bot_rows < 0) return fail(PARAPROX_ERR_INVALID_ARG, "negative reach or rows");
    if ((top_rows && !d_top) || (bot_rows && !d_bot)) return fail(PARAPROX_ERR_INVALID_ARG, "NULL halo source");
    paraprox_status st = check_image(img, false);
    if (st != PARAPROX_OK) return st;
    if (img->n != 1) return fail(PARAPROX_ERR_INVALID_ARG, "peer halos need n == 1");
    if ((top_rows || bot_rows) && src_pitch < img->w) return fail(PARAPROX_ERR_INVALID_ARG, "src_pitch < w");
    if (overlaps(d_in, d_out, img)) return fail(PARAPROX_ERR_INVALID_ARG, "d_out overlaps d_in");
    int dy, dx;
    scheme_reaches(scheme, reach, &dy, &dx);
    const Plan& p = get_plan(f, dy, dx);
    // a neighbour thinner than the halo would be clamped at its first row,
    // which is not the image's edge: refuse (dist.PeerStripe checks this too)
    if ((top_rows > 0 && top_rows < p.hy) || (bot_rows > 0 && bot_rows < p.hy))
        return fail(PARAPROX_ERR_INVALID_ARG, "neighbour rows fewer than the plan's halo h_y");
    const int ntop = std::min(top_rows, p.hy), nbot = std::min(bot_rows, p.hy);
    cudaStream_t cs = (cudaStream_t)s;
    const View v = view_of(img);
    if (ntop == 0 && nbot == 0) {  // nothing to read from the neighbours
        cudaError_t e = launch_stencil(p, d_in, v, d_out, img->pitch, (long long)img->h * img->pitch, cs);
        if (e != cudaSuccess) return cuda_fail(e, "stencil launch");
        return PARAPROX_OK;
    }
    bool taken = false;
    cudaError_t e = launch_stencil_peer(p, d_in, v, d_out, img->pitch, d_top + (long long)(top_rows - ntop) * src_pitch,
                                        ntop, d_bot, nbot, src_pitch, cs, &taken);
    if (e != cudaSuccess) return cuda_fail(e, "peer stencil launch");
    if (taken) return PARAPROX_OK;
    // fallback: gather the halo rows next to a copy of the stripe, then the
    // regular halo path (peer rows are read by the copy engine)
    const long long rows = (long long)ntop + img->h + nbot;
    DevBuf buf;
    buf.s = cs;
    PPX_CUDA(scratch_alloc(&buf.p, sizeof(float) * rows * img->w, cs));
    float* g = (float*)buf.p;
    const size_t rowb = sizeof(float) * img->w;
    if (ntop)
        PPX_CUDA(cudaMemcpy2DAsync(g, rowb, d_top + (long long)(top_rows - ntop) * src_pitch, sizeof(float) * src_pitch,
                                   rowb, ntop, cudaMemcpyDefault, cs));
    PPX_CUDA(cudaMemcpy2DAsync(g + (long long)ntop * img->w, rowb, d_in, sizeof(float) * img->pitch, rowb, img->h,
                               cudaMemcpyDefault, cs));
    if (nbot)
        PPX_CUDA(cudaMemcpy2DAsync(g + (long long)(ntop + img->h) * img->w, rowb, d_bot, sizeof(float) * src_pitch, rowb,
                                   nbot, cudaMemcpyDefault, cs));
    View vg;
    vg.n = 1;
    vg.h = img->h;
    vg.w = img->w;
    vg.pitch = img->w;
    vg.fstride = rows * img->w;
    vg.lo = -ntop;
    vg.hi = img->h - 1 + nbot;
    e = launch_stencil(p, g + (long long)ntop * img->w, vg, d_out, img->pitch, (long long)img->h * img->pitch, cs);
    if (e != cudaSuccess) return cuda_fail(e, "stencil launch");
    return PARAPROX_OK;
}

paraprox_status paraprox_ipc_export(const void* d_ptr, void* h_handle, long long* offset) {
    if (!d_ptr || !h_handle || !offset) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    static PFN_cuMemGetAddressRange_v3020 range = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            range = reinterpret_cast<PFN_cuMemGetAddressRange_v3020>(fn);
    });
    if (!range) return fail(PARAPROX_ERR_CUDA, "cuMemGetAddressRange unavailable");
    CUdeviceptr base = 0;
    size_t size = 0;
    if (range(&base, &size, (CUdeviceptr)d_ptr) != CUDA_SUCCESS) return fail(PARAPROX_ERR_CUDA, "cuMemGetAddressRange");
    cudaIpcMemHandle_t h;
    PPX_CUDA(cudaIpcGetMemHandle(&h, (void*)base));
    std::memcpy(h_handle, &h, sizeof(h));
    *offset = (long long)((CUdeviceptr)d_ptr - base);
    return PARAPROX_OK;
}

paraprox_status paraprox_ipc_open(const void* h_handle, void** d_base) {
    if (!h_handle || !d_base) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    cudaIpcMemHandle_t h;
    std::memcpy(&h, h_handle, sizeof(h));
    PPX_CUDA(cudaIpcOpenMemHandle(d_base, h, cudaIpcMemLazyEnablePeerAccess));
    return PARAPROX_OK;
}

paraprox_status paraprox_ipc_close(void* d_base) {
    if (!d_base) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    PPX_CUDA(cudaIpcCloseMemHandle(d_base));
    return PARAPROX_OK;
}

paraprox_status paraprox_hotspot_peer(const paraprox_hotspot_params* prm, paraprox_scheme scheme, int reach,
                                      const float* d_temp, const float* d_power, float* d_out,
                                      const paraprox_image* img, int steps, const float* d_top_temp,
                                      const float* d_top_power, int top_rows, const float* d_bot_temp,
                                      const float* d_bot_power, int bot_rows, long long src_pitch,
                                      paraprox_stream s) {
    if (!prm || !d_temp || !d_power || !d_out || !img) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (scheme < PARAPROX_EXACT || scheme > PARAPROX_CENTER) return fail(PARAPROX_ERR_INVALID_ARG, "unknown scheme");
    if (reach < 0 || steps < 1 || steps > kHotspotMaxSteps || top_rows < 0 || bot_rows < 0)
        return fail(PARAPROX_ERR_INVALID_ARG, "reach, steps (1..8) or rows out of range");
    if ((top_rows && (!d_top_temp || !d_top_power)) || (bot_rows && (!d_bot_temp || !d_bot_power)))
        return fail(PARAPROX_ERR_INVALID_ARG, "NULL halo source");
    paraprox_status st = check_image(img, false);
    if (st != PARAPROX_OK) return st;
    if (img->n != 1) return fail(PARAPROX_ERR_INVALID_ARG, "peer halos need n == 1");
    if ((top_rows || bot_rows) && src_pitch < img->w) return fail(PARAPROX_ERR_INVALID_ARG, "src_pitch < w");
    if (overlaps(d_temp, d_out, img) || overlaps(d_power, d_out, img))
        return fail(PARAPROX_ERR_INVALID_ARG, "d_out overlaps an input");
    const double c = prm->step_div_cap, gx = prm->rx_inv, gy = prm->ry_inv, gz = prm->rz_inv;
    paraprox_filter_s f;
    f.ky = f.kx = 3;
    f.separable = false;
    f.w = {0.f, (float)(c * gy), 0.f, (float)(c * gx), (float)(1.0 - 2.0 * c * gx - 2.0 * c * gy - c * gz),
           (float)(c * gx), 0.f, (float)(c * gy), 0.f};
    int dy, dx;
    scheme_reaches(scheme, reach, &dy, &dx);
    const Plan& p = get_plan(&f, dy, dx);
    cudaStream_t cs = (cudaStream_t)s;
    View v = view_of(img);
    const long long ofs = (long long)img->h * img->pitch;
    if (p.hy == 0 && p.hx == 0) {  // centre at full reach: no neighbour read, fused steps
        Addend add;
        add.p = d_power;
        add.pitch = img->pitch;
        add.fstride = ofs;
        add.alpha = (float)c;
        add.beta = (float)(c * gz * prm->t_amb);
        add.steps = steps;
        cudaError_t e = launch_stencil(p, d_temp, v, d_out, img->pitch, ofs, cs, &add);
        if (e != cudaSuccess) return cuda_fail(e, "hotspot fused steps");
        return PARAPROX_OK;
    }
    const int need = steps * p.hy;  // halo rows of `steps` steps
    HotspotPeer peer;
    peer.ntop = top_rows ? need : 0;
    peer.nbot = bot_rows ? need : 0;
    if ((top_rows && top_rows < need) || (bot_rows && bot_rows < need))
        return fail(PARAPROX_ERR_INVALID_ARG, "fewer halo rows than steps x plan halo");
    peer.top_t = top_rows ? d_top_temp + (long long)(top_rows - need) * src_pitch : nullptr;
    peer.top_p = top_rows ? d_top_power + (long long)(top_rows - need) * src_pitch : nullptr;
    peer.bot_t = d_bot_temp;
    peer.bot_p = d_bot_power;
    peer.pitch = src_pitch;
    cudaError_t e = launch_hotspot_tb(p, d_temp, d_power, d_out, v, ofs, (float)c, (float)(c * gz * prm->t_amb), steps,
                                      cs, &peer);
    if (e != cudaSuccess) return cuda_fail(e, "hotspot peer pass");
    return PARAPROX_OK;
}

paraprox_status paraprox_flag_wait(const long long* d_flag, long long target, paraprox_stream s) {
    if (!d_flag) return fail(PARAPROX_ERR_INVALID_ARG, "NULL flag");
    PPX_CUDA(launch_flag_wait(d_flag, target, (cudaStream_t)s));
    return PARAPROX_OK;
}

paraprox_status paraprox_flag_set(long long* d_flag, long long value, paraprox_stream s) {
    if (!d_flag) return fail(PARAPROX_ERR_INVALID_ARG, "NULL flag");
    PPX_CUDA(launch_flag_set(d_flag, value, (cudaStream_t)s));
    return PARAPROX_OK;
}

paraprox_status paraprox_quality(const float* d_exact, const float* d_approx, const paraprox_image* img,
                                 paraprox_metric m, double* h_quality, paraprox_stream s) {
    if (!h_quality) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    double p3[3];
    paraprox_status st = quality_partials_impl(d_exact, d_approx, img, m, p3, s);
    if (st != PARAPROX_OK) return st;
    *h_quality = quality_of(p3, m);
    return PARAPROX_OK;
}

paraprox_status paraprox_quality_partials(const float* d_exact, const float* d_approx, const paraprox_image* img,
                                          paraprox_metric m, double* h_partials3, paraprox_stream s) {
    return quality_partials_impl(d_exact, d_approx, img, m, h_partials3, s);
}

paraprox_status paraprox_quality_partials_async(const float* d_exact, const float* d_approx,
                                                const paraprox_image* img, paraprox_metric m, double* d_partials3,
                                                paraprox_stream s) {
    if (!d_exact || !d_approx || !d_partials3) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (!metric_ok(m)) return fail(PARAPROX_ERR_INVALID_ARG, "unknown metric");
    paraprox_status st = check_image(img, false);
    if (st != PARAPROX_OK) return st;
    cudaStream_t cs = (cudaStream_t)s;
    DevBuf buf;
    buf.s = cs;
    PPX_CUDA(scratch_alloc(&buf.p, sizeof(double) * quality_scratch_doubles((long long)img->n * img->h * img->w), cs));
    cudaError_t err = launch_quality(d_exact, d_approx, view_of(img), m, d_partials3, (double*)buf.p, cs);
    if (err != cudaSuccess) return cuda_fail(err, "quality launch");
    return PARAPROX_OK;
}

paraprox_status paraprox_quality_from_partials(const double* h_partials3, paraprox_metric m, double* h_quality) {
    if (!h_partials3 || !h_quality) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (!metric_ok(m)) return fail(PARAPROX_ERR_INVALID_ARG, "unknown metric");
    *h_quality = quality_of(h_partials3, m);
    return PARAPROX_OK;
}

paraprox_status paraprox_tune_candidates(paraprox_filter f, int cap, int* n, paraprox_scheme* schemes,
                                         int* reaches) {
    if (!f || !n) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (cap < 0) return fail(PARAPROX_ERR_INVALID_ARG, "cap < 0");
    std::vector<Candidate> c = candidates(f);
    *n = (int)c.size();
    for (int k = 0; k < (int)c.size() && k < cap; ++k) {
        if (schemes) schemes[k] = c[k].scheme;
        if (reaches) reaches[k] = c[k].reach;
    }
    return PARAPROX_OK;
}

paraprox_status paraprox_tune_candidates_ex(paraprox_filter f, int flags, int cap, int* n, paraprox_scheme* schemes,
                                            int* reaches) {
    if (!f || !n) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (cap < 0) return fail(PARAPROX_ERR_INVALID_ARG, "cap < 0");
    if (flags < 1 || flags > 3) return fail(PARAPROX_ERR_INVALID_ARG, "flags not in 1..3");
    std::vector<Candidate> c = candidates_ex(f, flags);
    *n = (int)c.size();
    for (int k = 0; k < (int)c.size() && k < cap; ++k) {
        if (schemes) schemes[k] = c[k].scheme;
        if (reaches) reaches[k] = c[k].reach;
    }
    return PARAPROX_OK;
}

paraprox_status paraprox_tune_partials_ex(paraprox_filter f, int flags, const float* d_train,
                                          const paraprox_image* img, paraprox_metric m, double* h_partials,
                                          paraprox_stream s) {
    if (!f) return fail(PARAPROX_ERR_INVALID_ARG, "filter is NULL");
    if (flags < 1 || flags > 3) return fail(PARAPROX_ERR_INVALID_ARG, "flags not in 1..3");
    return tune_partials_impl(f, d_train, img, m, candidates_ex(f, flags), h_partials, s);
}

paraprox_status paraprox_tune_decide_ex(paraprox_filter f, int flags, const double* h_partials, paraprox_metric m,
                                        double toq, paraprox_scheme* out_scheme, int* out_reach,
                                        double* out_quality) {
    if (!f || !out_scheme || !out_reach || !out_quality) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (flags < 1 || flags > 3) return fail(PARAPROX_ERR_INVALID_ARG, "flags not in 1..3");
    paraprox_status st = check_toq(toq, m);
    if (st != PARAPROX_OK) return st;
    std::vector<Candidate> c = candidates_ex(f, flags);
    if (!h_partials && !c.empty()) return fail(PARAPROX_ERR_INVALID_ARG, "NULL partials");
    return decide(c, h_partials, m, toq, out_scheme, out_reach, out_quality);
}

paraprox_status paraprox_tune_ex(paraprox_filter f, int flags, const float* d_train, const paraprox_image* img,
                                 double toq, paraprox_metric m, paraprox_scheme* out_scheme, int* out_reach,
                                 double* out_quality, paraprox_stream s) {
    if (!f || !out_scheme || !out_reach || !out_quality) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (flags < 1 || flags > 3) return fail(PARAPROX_ERR_INVALID_ARG, "flags not in 1..3");
    paraprox_status st = check_toq(toq, m);
    if (st != PARAPROX_OK) return st;
    std::vector<Candidate> c = candidates_ex(f, flags);
    std::vector<double> parts(3 * c.size() + 3);
    st = tune_partials_impl(f, d_train, img, m, c, parts.data(), s, toq);
    if (st != PARAPROX_OK) return st;
    return decide(c, parts.data(), m, toq, out_scheme, out_reach, out_quality);
}

paraprox_status paraprox_tune_partials(paraprox_filter f, const float* d_train, const paraprox_image* img,
                                       paraprox_metric m, double* h_partials, paraprox_stream s) {
    if (!f) return fail(PARAPROX_ERR_INVALID_ARG, "filter is NULL");
    return tune_partials_impl(f, d_train, img, m, candidates(f), h_partials, s);
}

paraprox_status paraprox_tune_decide(paraprox_filter f, const double* h_partials, paraprox_metric m, double toq,
                                     paraprox_scheme* out_scheme, int* out_reach, double* out_quality) {
    if (!f || !out_scheme || !out_reach || !out_quality) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    paraprox_status st = check_toq(toq, m);
    if (st != PARAPROX_OK) return st;
    std::vector<Candidate> c = candidates(f);
    if (!c.empty() && !h_partials) return fail(PARAPROX_ERR_INVALID_ARG, "NULL partials");
    return decide(c, h_partials, m, toq, out_scheme, out_reach, out_quality);
}

paraprox_status paraprox_tune(paraprox_filter f, const float* d_train, const paraprox_image* img, double toq,
                              paraprox_metric m, paraprox_scheme* out_scheme, int* out_reach,
                              double* out_quality, paraprox_stream s) {
    if (!f || !out_scheme || !out_reach || !out_quality) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    paraprox_status st = check_toq(toq, m);
    if (st != PARAPROX_OK) return st;
    std::vector<Candidate> c = candidates(f);
    std::vector<double> parts(3 * c.size() + 3);
    st = tune_partials_impl(f, d_train, img, m, c, parts.data(), s, toq);
    if (st != PARAPROX_OK) return st;
    return decide(c, parts.data(), m, toq, out_scheme, out_reach, out_quality);
}

paraprox_status paraprox_run_host(paraprox_filter f, paraprox_scheme scheme, int reach, const float* h_in,
                                  float* h_out, const paraprox_image* img, paraprox_stream s) {
    if (!f || !h_in || !h_out) return fail(PARAPROX_ERR_INVALID_ARG, "NULL pointer");
    if (scheme < PARAPROX_EXACT || scheme > PARAPROX_SKIP_BOTH) return fail(PARAPROX_ERR_INVALID_ARG, "unknown scheme");
    if (reach < (is_skip_scheme(scheme) ? 1 : 0)) return fail(PARAPROX_ERR_INVALID_ARG, "reach < 0 or rate < 1");
    paraprox_status st = check_image(img, false);
    if (st != PARAPROX_OK) return st;
    if (overlaps(h_in, h_out, img)) return fail(PARAPROX_ERR_INVALID_ARG, "h_out overlaps h_in");
    int dy, dx;
    if (is_skip_scheme(scheme)) scheme_skips(scheme, reach, &dy, &dx);
    else scheme_reaches(scheme, reach, &dy, &dx);
    const Plan& p = is_skip_scheme(scheme) ? get_plan_skip(f, dy, dx) : get_plan(f, dy, dx);
    cudaStream_t cs = (cudaStream_t)s;
    const int n = img->n, h = img->h, w = img->w;
    const long long plane = (long long)h * w;
    const long long hfs = n > 1 ? img->frame_stride : 0;
    DevBuf buf;
    buf.s = cs;
    PPX_CUDA(scratch_alloc(&buf.p, sizeof(float) * 2 * plane * n, cs));
    float* din = (float*)buf.p;
    float* dout = din + plane * n;
    // chunks: frames when batched, else row bands of >= 64 rows (halo rows
    // come along).  ~8 MiB per chunk, at most 64: each chunk costs ~30 us of
    // host calls (2 MiB chunks made c2's 64 MiB 30 % slower than 8 MiB ones).
    // The pipeline's fill (first upload) and drain (last download) are not
    // overlapped, so the chunks ramp up and down (1/8, 1/4, 1/2 of the target
    // at both ends) when there is room: uniform 8 MiB chunks left c2's 64 MiB
    // at ~0.8 of the PCIe duplex bound.
    const long long units = n > 1 ? n : h;
    const long long unit_bytes = (long long)sizeof(float) * (n > 1 ? plane : w);
    const long long min_units = n > 1 ? 1 : std::min<long long>(h, 64);
    long long target = std::max(min_units, (8LL << 20) / std::max(1LL, unit_bytes));
    target = std::max(target, (units + 63) / 64);
    std::vector<long long> bounds(1, 0);
    {
        const long long r[3] = {std::max(min_units, target / 8), std::max(min_units, target / 4),
                                std::max(min_units, target / 2)};
        const long long ramp = r[0] + r[1] + r[2];
        if (2 * ramp + target <= units && target > r[2]) {
            for (long long q : r) bounds.push_back(bounds.back() + q);
            const long long mid = units - 2 * ramp;
            const long long nm = std::max(1LL, (mid + target - 1) / target);
            const long long b0 = bounds.back();
            for (long long c = 1; c <= nm; ++c) bounds.push_back(b0 + mid * c / nm);
            for (int k = 2; k >= 0; --k) bounds.push_back(bounds.back() + r[k]);
        } else {
            const long long nc = std::max(1LL, std::min(units / min_units, (units + target - 1) / target));
            for (long long c = 1; c <= nc; ++c) bounds.push_back(units * c / nc);
        }
    }
    const int chunks = (int)bounds.size() - 1;
    // copy streams and events are created once per thread and device, reused
    struct Pipe {
        int dev = -1;
        cudaStream_t up = nullptr, down = nullptr;
        std::vector<cudaEvent_t> ev;
    };
    static thread_local Pipe pipe;
    int dev = 0;
    PPX_CUDA(cudaGetDevice(&dev));
    if (pipe.dev != dev) {
        if (pipe.up) cudaStreamDestroy(pipe.up);
        if (pipe.down) cudaStreamDestroy(pipe.down);
        for (auto& e : pipe.ev) cudaEventDestroy(e);
        pipe = Pipe();
        PPX_CUDA(cudaStreamCreateWithFlags(&pipe.up, cudaStreamNonBlocking));
        PPX_CUDA(cudaStreamCreateWithFlags(&pipe.down, cudaStreamNonBlocking));
        pipe.dev = dev;
    }
    while ((int)pipe.ev.size() < 3 * chunks + 1) {
        cudaEvent_t e;
        PPX_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        pipe.ev.push_back(e);
    }
    cudaStream_t up = pipe.up, down = pipe.down;
    std::vector<cudaEvent_t>& ev = pipe.ev;
    cudaError_t err = cudaSuccess;
    auto bail = [&](cudaError_t e2, const char* where) {
        cudaStreamSynchronize(down);
        cudaStreamSynchronize(up);
        return cuda_fail(e2, where);
    };
    const bool frames_contig = img->pitch == w && hfs == plane;
    // the device scratch is stream-ordered on cs: make the copy streams wait for it
    if ((err = cudaEventRecord(ev[3 * chunks], cs)) != cudaSuccess) return bail(err, "record");
    if ((err = cudaStreamWaitEvent(up, ev[3 * chunks], 0)) != cudaSuccess) return bail(err, "wait");
    const size_t rowb = sizeof(float) * w;
    int copied = 0;  // rows of the single frame already uploaded
    for (int c = 0; c < chunks; ++c) {
        View v;
        const float* kin;
        float* kout;
        if (n > 1) {
            const int f0 = (int)bounds[c], f1 = (int)bounds[c + 1];
            if (frames_contig) {
                if ((err = cudaMemcpyAsync(din + f0 * plane, h_in + f0 * plane, sizeof(float) * plane * (f1 - f0),
                                           cudaMemcpyHostToDevice, up)) != cudaSuccess)
                    return bail(err, "H2D");
            } else {
                for (int fr = f0; fr < f1; ++fr)
                    if ((err = cudaMemcpy2DAsync(din + fr * plane, rowb, h_in + fr * hfs, sizeof(float) * img->pitch,
                                                 rowb, h, cudaMemcpyHostToDevice, up)) != cudaSuccess)
                        return bail(err, "H2D");
            }
            v = {f1 - f0, h, w, (long long)w, plane, 0, h - 1};
            kin = din + f0 * plane;
            kout = dout + f0 * plane;
        } else {
            const int r0 = (int)bounds[c], r1 = (int)bounds[c + 1];
            const int need = std::min(h, r1 + p.hy);
            if (need > copied) {
                if ((err = cudaMemcpy2DAsync(din + (long long)copied * w, rowb, h_in + (long long)copied * img->pitch,
                                             sizeof(float) * img->pitch, rowb, need - copied,
                                             cudaMemcpyHostToDevice, up)) != cudaSuccess)
                    return bail(err, "H2D");
                copied = need;
            }
            v = {1, r1 - r0, w, (long long)w, (long long)(r1 - r0) * w, -r0, need - 1 - r0};
            kin = din + (long long)r0 * w;
            kout = dout + (long long)r0 * w;
        }
        if ((err = cudaEventRecord(ev[3 * c], up)) != cudaSuccess) return bail(err, "record");
        if ((err = cudaStreamWaitEvent(cs, ev[3 * c], 0)) != cudaSuccess) return bail(err, "wait");
        err = launch_stencil(p, kin, v, kout, w, v.n > 1 ? plane : (long long)v.h * w, cs);
        if (err != cudaSuccess) return bail(err, "stencil launch");
        if ((err = cudaEventRecord(ev[3 * c + 1], cs)) != cudaSuccess) return bail(err, "record");
        if ((err = cudaStreamWaitEvent(down, ev[3 * c + 1], 0)) != cudaSuccess) return bail(err, "wait");
        if (n > 1) {
            const int f0 = (int)bounds[c], f1 = (int)bounds[c + 1];
            if (frames_contig) {
                if ((err = cudaMemcpyAsync(h_out + f0 * plane, dout + f0 * plane, sizeof(float) * plane * (f1 - f0),
                                           cudaMemcpyDeviceToHost, down)) != cudaSuccess)
                    return bail(err, "D2H");
            } else {
                for (int fr = f0; fr < f1; ++fr)
                    if ((err = cudaMemcpy2DAsync(h_out + fr * hfs, sizeof(float) * img->pitch, dout + fr * plane, rowb,
                                                 rowb, h, cudaMemcpyDeviceToHost, down)) != cudaSuccess)
                        return bail(err, "D2H");
            }
        } else {
            const int r0 = (int)bounds[c], r1 = (int)bounds[c + 1];
            if ((err = cudaMemcpy2DAsync(h_out + (long long)r0 * img->pitch, sizeof(float) * img->pitch,
                                         dout + (long long)r0 * w, rowb, rowb, r1 - r0, cudaMemcpyDeviceToHost,
                                         down)) != cudaSuccess)
                return bail(err, "D2H");
        }
    }
    // the scratch is freed on cs: order it after the last download
    if ((err = cudaEventRecord(ev[3 * chunks - 1], down)) != cudaSuccess) return bail(err, "record");
    if ((err = cudaStreamWaitEvent(cs, ev[3 * chunks - 1], 0)) != cudaSuccess) return bail(err, "wait");
    err = cudaStreamSynchronize(down);
    if (err != cudaSuccess) return bail(err, "D2H sync");
    buf.p = nullptr;
    PPX_CUDA(cudaFreeAsync(din, cs));
    PPX_CUDA(cudaStreamSynchronize(cs));
    return PARAPROX_OK;
}

const char* paraprox_status_string(paraprox_status st) {
    switch (st) {
    case PARAPROX_OK: return "ok";
    case PARAPROX_ERR_INVALID_ARG: return "invalid argument";
    case PARAPROX_ERR_UNSUPPORTED: return "unsupported";
    case PARAPROX_ERR_CUDA: return "CUDA error";
    case PARAPROX_ERR_ALLOC: return "allocation failed";
    default: return "unknown status";
    }
}

const char* paraprox_last_error(void) { return t_err.c_str(); }
int paraprox_version(void) { return PARAPROX_VERSION; }
unsigned long long paraprox_launch_count(void) { return g_launches.load(); }
const char* paraprox_last_kernel(void) { return t_last_kernel; }

}  // extern "C"
