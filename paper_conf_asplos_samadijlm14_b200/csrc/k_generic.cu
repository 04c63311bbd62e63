// k_generic.cu -- the fallback stencil kernel: any filter shape up to 17x17,
// any index maps, any pitch/alignment.  One thread per output, taps from a
// kernel-parameter table, clamped __ldg loads through L1/L2.  Correct for every
// case the fast kernels (k_dense.cu, k_sep.cu) do not take; never a CPU path.
#include "internal.h"

namespace ppx {

struct TapTable {
    int n;
    signed char oy[kMaxTaps];
    signed char ox[kMaxTaps];
    float w[kMaxTaps];
};

__global__ void __launch_bounds__(256) k_stencil_generic(const float* __restrict__ in, View v,
                                                         float* __restrict__ out, long long opitch,
                                                         long long ofs, const __grid_constant__ TapTable t,
                                                         const Addend add) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x;
    if (x >= v.w) return;
    // grid-stride over rows and frames: any h, n the ABI accepts launches
    for (int y = blockIdx.y * blockDim.y + threadIdx.y; y < v.h; y += gridDim.y * blockDim.y)
    for (int f = blockIdx.z; f < v.n; f += gridDim.z) {
        const float* F = in + (long long)f * v.fstride;
        float acc = 0.f;
        for (int k = 0; k < t.n; ++k) {
            const int yy = min(max(y + (int)t.oy[k], v.lo), v.hi);
            const int xx = min(max(x + (int)t.ox[k], 0), v.w - 1);
            acc = fmaf(t.w[k], __ldg(F + (long long)yy * v.pitch + xx), acc);
        }
        if (add.p) {
            const float a = add.p[(long long)f * add.fstride + (long long)y * add.pitch + x];
            acc = __fadd_rn(__fmaf_rn(add.alpha, a, acc), add.beta);
            // fused steps of a centre-only plan (one tap at (0, 0)), as k_pointwise
            for (int k = 1; k < add.steps; ++k)
                acc = __fadd_rn(__fmaf_rn(add.alpha, a, __fmaf_rn(t.w[0], acc, 0.f)), add.beta);
        }
        out[(long long)f * ofs + (long long)y * opitch + x] = acc;
    }
}

// Folded taps in (row rep, column rep) ascending order.  Separable plans are
// expanded to their outer product here (the fused kernel keeps them apart).
static void fill_taps(const Plan& p, TapTable* t) {
    t->n = 0;
    for (int a = 0; a < p.ny; ++a)
        for (int b = 0; b < p.nx; ++b) {
            t->oy[t->n] = (signed char)p.ay[a];
            t->ox[t->n] = (signed char)p.ax[b];
            t->w[t->n] = p.separable ? p.wyf[a] * p.wxf[b] : p.wf[a * p.nx + b];
            ++t->n;
        }
}

cudaError_t launch_generic(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                           long long ofs, cudaStream_t s, const Addend* add) {
    TapTable t;
    fill_taps(p, &t);
    dim3 block(32, 8);
    const int gy = (v.h + 7) / 8;
    dim3 grid((v.w + 31) / 32, gy < 65535 ? gy : 65535, v.n < 65535 ? v.n : 65535);
    k_stencil_generic<<<grid, block, 0, s>>>(in, v, out, opitch, ofs, t, add ? *add : Addend());
    count_launch("generic");
    return cudaGetLastError();
}

}  // namespace ppx
