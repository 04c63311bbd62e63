// quality.cuh -- per-thread accumulation of the output-quality terms (Table 1
// metrics) and the deterministic block reduction, shared
// by the quality kernels (k_quality.cu) and the fused stencil + quality
// epilogues of the tile and map kernels (the tuner's candidates, the runtime's
// checks).
#pragma once

#include "internal.h"

namespace ppx {

// Per-thread accumulators.  L2 / PSNR: fp64 (the difference of two fp32
// values is exact in fp64; 2 DFMA per pixel).  MRE needs a quotient per
// pixel, and fp64 division is far below the HBM rate on this part (the first
// version ran at ~1.5 TB/s), so each term |A-E|/|E| is formed as an unevaluated
// fp32 pair q0 + q1 (exact difference by TwoSum, quotient by the approximate
// fp32 reciprocal plus one FMA remainder correction, relative error ~2^-46)
// whose two parts are summed in two fp64 accumulators.  Terms the pair arithmetic cannot carry (|E| tiny, |A-E| huge) take
// the fp64 path.  Tests bound the result against the fp64 oracle at 1e-12.
template <int M>
struct QAcc {
    double s0 = 0.0, s1 = 0.0;
    bool bad = false;                                       // never set: no fix-up pass
    __device__ __forceinline__ void reset() {}
    __device__ __forceinline__ void fix(float, float) {}
    __device__ __forceinline__ void add(float e, float a) {
        const double de = (double)e, da = (double)a;
        const double d = da - de;
        if (M == PARAPROX_L2) {
            s0 = fma(d, d, s0);
            s1 = fma(de, de, s1);
        } else {
            s0 = fma(d, d, s0);
        }
    }
    __device__ __forceinline__ void get(double& a, double& b) const {
        a = s0;
        b = s1;
    }
};

__device__ __forceinline__ void two_sum(float a, float b, float& s, float& err) {
    s = __fadd_rn(a, b);
    const float bb = __fsub_rn(s, a);
    err = __fadd_rn(__fsub_rn(a, __fsub_rn(s, bb)), __fsub_rn(b, bb));
}

__device__ __forceinline__ float rcp_approx(float x) {
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    return r;
}

template <>
struct QAcc<PARAPROX_MRE> {
    double hi = 0.0, lo = 0.0;  // sums of the leading and trailing parts of the terms
    bool bad = false;  // some term the pair arithmetic cannot carry was seen
    // the fast path needs |E| in [1e-30, 1e30] and |A-E| <= 1e30 (and E != 0,
    // the S12 convention); a CTA that saw any other term redoes all of its
    // terms in fp64 (fix pass), so the fast path carries no per-term select
    __device__ __forceinline__ static bool fast_ok(float ae, float dh) {
        return ae >= 1e-30f && ae <= 1e30f && fabsf(dh) <= 1e30f;
    }
    __device__ __forceinline__ void add(float e, float a) {
        float dh, dl;
        two_sum(a, -e, dh, dl);  // A - E exactly, as dh + dl
        const float ae = fabsf(e);
        bad |= !fast_ok(ae, dh);
        // q0 + q1 = (A-E) / |E| to ~2^-46: the remainder of the first quotient
        // is exact under the FMA, so the approximate reciprocal's own error is
        // corrected by the second term; the term |q0 + q1| = |q0| + q1 * sgn(q0)
        // (|q1| << |q0|, and q0 = 0 only when A = E)
        const float rc = rcp_approx(ae);
        const float q0 = __fmul_rn(dh, rc);
        const float rem = __fadd_rn(__fmaf_rn(-q0, ae, dh), dl);
        hi += (double)fabsf(q0);
        const float q1 = __fmul_rn(rem, rc);
        lo += (double)__uint_as_float(__float_as_uint(q1) ^ (__float_as_uint(q0) & 0x80000000u));  // q1 * sgn(q0)
    }
    // fix pass: every term of the CTA again, in fp64
    __device__ __forceinline__ void reset() { hi = lo = 0.0; }
    __device__ __forceinline__ void fix(float e, float a) {
        const double de = (double)e, da = (double)a;
        hi += de != 0.0 ? fabs(da - de) / fabs(de) : (da == 0.0 ? 0.0 : 1.0);
    }
    __device__ __forceinline__ void get(double& a, double& b) const {
        a = hi + lo;
        b = 0.0;
    }
};

__device__ __forceinline__ void block_sum2(double& s0, double& s1) {
    __shared__ double red[2][32];
    for (int o = 16; o > 0; o >>= 1) {
        s0 += __shfl_down_sync(0xffffffffu, s0, o);
        s1 += __shfl_down_sync(0xffffffffu, s1, o);
    }
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (lane == 0) {
        red[0][warp] = s0;
        red[1][warp] = s1;
    }
    __syncthreads();
    if (warp == 0) {
        const int nw = blockDim.x >> 5;
        s0 = lane < nw ? red[0][lane] : 0.0;
        s1 = lane < nw ? red[1][lane] : 0.0;
        for (int o = 16; o > 0; o >>= 1) {
            s0 += __shfl_down_sync(0xffffffffu, s0, o);
            s1 += __shfl_down_sync(0xffffffffu, s1, o);
        }
    }
}

// Runtime-metric accumulator of the fused epilogues: same terms as QAcc (MRE
// in the fp32-pair form, the rare terms it cannot carry inline in fp64; L2 and
// PSNR in fp64).  get() returns the two partials k_quality_final expects.
struct RAcc {
    double a = 0.0, b = 0.0;
    __device__ __forceinline__ void add(int m, float e, float x) {
        if (m == PARAPROX_MRE) {
            float dh, dl;
            two_sum(x, -e, dh, dl);
            const float ae = fabsf(e);
            if (QAcc<PARAPROX_MRE>::fast_ok(ae, dh)) {
                if (dh < 0.f) {
                    dh = -dh;
                    dl = -dl;
                }
                const float rc = rcp_approx(ae);
                const float q0 = __fmul_rn(dh, rc);
                const float rem = __fadd_rn(__fmaf_rn(-q0, ae, dh), dl);
                a += (double)q0;
                b += (double)__fmul_rn(rem, rc);
            } else {
                const double de = (double)e, dx = (double)x;
                a += de != 0.0 ? fabs(dx - de) / fabs(de) : (dx == 0.0 ? 0.0 : 1.0);
            }
        } else {
            const double de = (double)e, d = (double)x - de;
            a = fma(d, d, a);
            if (m == PARAPROX_L2) b = fma(de, de, b);
        }
    }
    __device__ __forceinline__ void get(int m, double& s0, double& s1) const {
        if (m == PARAPROX_MRE) {
            s0 = a + b;
            s1 = 0.0;
        } else {
            s0 = a;
            s1 = b;
        }
    }
};

}  // namespace ppx
