// k_quality.cu -- output-quality partial sums (Table 1
// metrics): mean relative error, L2-norm, PSNR.
//
// fp32 inputs; fp64 per-thread sums (MRE terms formed as fp32 pairs), fp64
// reductions.  Deterministic: a fixed number of CTAs
// (kQualityBlocks, or fewer rows), each walking its rows in a fixed order,
// fixed warp-shuffle trees, then one CTA summing the per-CTA partials in a
// fixed order.  No atomics.  8 bytes of HBM read per pixel, nothing written.
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
    bool bad = false;  // a term the pair arithmetic cannot carry was skipped
    // the fast path skips terms with |E| tiny or huge or |A-E| huge (and the
    // E == 0 convention, S12); a second pass adds exactly those in fp64
    __device__ __forceinline__ static bool fast_ok(float ae, float dh) {
        return ae >= 1e-30f && ae <= 1e30f && fabsf(dh) <= 1e30f;
    }
    __device__ __forceinline__ void add(float e, float a) {
        float dh, dl;
        two_sum(a, -e, dh, dl);  // A - E exactly, as dh + dl
        const float ae = fabsf(e);
        const bool ok = fast_ok(ae, dh);
        bad |= !ok;
        if (dh < 0.f) {
            dh = -dh;
            dl = -dl;
        }
        // q0 + q1 = |A-E| / |E| to ~2^-46: the remainder of the first quotient
        // is exact under the FMA, so the approximate reciprocal's own error is
        // corrected by the second term
        const float rc = rcp_approx(ae);
        const float q0 = __fmul_rn(dh, rc);
        const float rem = __fadd_rn(__fmaf_rn(-q0, ae, dh), dl);
        hi += ok ? (double)q0 : 0.0;
        lo += ok ? (double)__fmul_rn(rem, rc) : 0.0;
    }
    __device__ __forceinline__ void fix(float e, float a) {
        float dh, dl;
        two_sum(a, -e, dh, dl);
        if (!fast_ok(fabsf(e), dh)) {
            const double de = (double)e, da = (double)a;
            hi += de != 0.0 ? fabs(da - de) / fabs(de) : (da == 0.0 ? 0.0 : 1.0);
        }
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

// Contiguous images (pitch == w, frames back to back) are one flat array:
// each thread keeps kQU independent 128-bit loads of E and of A in flight per
// iteration (grid-stride, fixed grid), so the HBM pipe stays full while the
// fp64 division chain of MRE runs.  Other layouts walk rows.
constexpr int kQU = 4;

template <int M>
__global__ void __launch_bounds__(256, M == PARAPROX_MRE ? 3 : 2) k_quality_flat(const float* __restrict__ E, const float* __restrict__ A,
                                                      long long count, double* __restrict__ part) {
    QAcc<M> q;
    const long long n4 = count >> 2;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const float4* e4 = reinterpret_cast<const float4*>(E);
    const float4* a4 = reinterpret_cast<const float4*>(A);
    auto sweep = [&](auto&& op) {
        for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += kQU * stride) {
            float4 e[kQU], a[kQU];
#pragma unroll
            for (int u = 0; u < kQU; ++u) {
                const long long j = i + u * stride;
                if (j < n4) {
                    e[u] = __ldcs(e4 + j);
                    a[u] = __ldcs(a4 + j);
                } else {
                    e[u] = a[u] = make_float4(1.f, 1.f, 1.f, 1.f);  // |1-1|/|1| = 0, (1-1)^2 = 0
                }
            }
#pragma unroll
            for (int u = 0; u < kQU; ++u) {
                if (i + u * stride >= n4) continue;
                op(e[u].x, a[u].x);
                op(e[u].y, a[u].y);
                op(e[u].z, a[u].z);
                op(e[u].w, a[u].w);
            }
        }
        if (blockIdx.x == 0)
            for (long long x = (n4 << 2) + threadIdx.x; x < count; x += blockDim.x) op(E[x], A[x]);
    };
    sweep([&](float e, float a) { q.add(e, a); });
    if constexpr (M == PARAPROX_MRE)
        if (__syncthreads_or(q.bad)) sweep([&](float e, float a) { q.fix(e, a); });
    double s0, s1;
    q.get(s0, s1);
    block_sum2(s0, s1);
    if (threadIdx.x == 0) {
        part[2 * blockIdx.x] = s0;
        part[2 * blockIdx.x + 1] = s1;
    }
}

template <int M>
__global__ void __launch_bounds__(256, M == PARAPROX_MRE ? 3 : 2) k_quality_partials(const float* __restrict__ E,
                                                          const float* __restrict__ A, View v,
                                                          double* __restrict__ part) {
    QAcc<M> q;
    const long long rows = (long long)v.n * v.h;
    const bool vec = ((v.pitch & 3) == 0) && ((v.fstride & 3) == 0) &&
                     ((((uintptr_t)E) | ((uintptr_t)A)) & 15) == 0;
    const int w4 = vec ? (v.w >> 2) : 0;
    auto sweep = [&](auto&& op) {
        for (long long R = blockIdx.x; R < rows; R += gridDim.x) {
            const long long f = R / v.h, y = R - f * v.h;
            const long long off = f * v.fstride + y * v.pitch;
            const float4* e4 = reinterpret_cast<const float4*>(E + off);
            const float4* a4 = reinterpret_cast<const float4*>(A + off);
            for (int x = threadIdx.x; x < w4; x += kQU * blockDim.x) {
                float4 e[kQU], a[kQU];
#pragma unroll
                for (int u = 0; u < kQU; ++u) {
                    const int j = x + u * blockDim.x;
                    if (j < w4) {
                        e[u] = __ldcs(e4 + j);
                        a[u] = __ldcs(a4 + j);
                    } else {
                        e[u] = a[u] = make_float4(1.f, 1.f, 1.f, 1.f);
                    }
                }
#pragma unroll
                for (int u = 0; u < kQU; ++u) {
                    if (x + u * (int)blockDim.x >= w4) continue;
                    op(e[u].x, a[u].x);
                    op(e[u].y, a[u].y);
                    op(e[u].z, a[u].z);
                    op(e[u].w, a[u].w);
                }
            }
            for (int x = (w4 << 2) + threadIdx.x; x < v.w; x += blockDim.x) op(__ldcs(E + off + x), __ldcs(A + off + x));
        }
    };
    sweep([&](float e, float a) { q.add(e, a); });
    if constexpr (M == PARAPROX_MRE)
        if (__syncthreads_or(q.bad)) sweep([&](float e, float a) { q.fix(e, a); });
    double s0, s1;
    q.get(s0, s1);
    block_sum2(s0, s1);
    if (threadIdx.x == 0) {
        part[2 * blockIdx.x] = s0;
        part[2 * blockIdx.x + 1] = s1;
    }
}

template <int M>
__global__ void __launch_bounds__(1024) k_quality_final(const double* __restrict__ part, int g,
                                                        double count, double* __restrict__ out3) {
    double s0 = 0.0, s1 = 0.0;
    for (int k = threadIdx.x; k < g; k += blockDim.x) {
        s0 += part[2 * k];
        s1 += part[2 * k + 1];
    }
    block_sum2(s0, s1);
    if (threadIdx.x == 0) {
        if (M == PARAPROX_L2) {
            out3[0] = s0;
            out3[1] = s1;
            out3[2] = count;
        } else {
            out3[0] = s0;
            out3[1] = count;
            out3[2] = 0.0;
        }
    }
}

// d_scratch: >= 2 * kQualityBlocks doubles.  Writes 3 doubles at d_part3.
cudaError_t launch_quality(const float* e, const float* a, const View& v, paraprox_metric m,
                           double* d_part3, double* d_scratch, cudaStream_t s) {
    const long long rows = (long long)v.n * v.h;
    const double count = (double)v.n * (double)v.h * (double)v.w;
    const bool flat = v.pitch == v.w && (v.n == 1 || v.fstride == (long long)v.h * v.w) &&
                      ((((uintptr_t)e) | ((uintptr_t)a)) & 15) == 0;
    const long long cnt = (long long)v.n * v.h * v.w;
    int g;
    if (flat) {
        const long long chunks = (cnt / 4 + 255) / 256;
        g = (int)(chunks < kQualityBlocks ? (chunks > 0 ? chunks : 1) : kQualityBlocks);
    } else {
        g = (int)(rows < kQualityBlocks ? rows : kQualityBlocks);
    }
#define PPX_QUALITY_CASE(M)                                                                    \
    if (flat) k_quality_flat<M><<<g, 256, 0, s>>>(e, a, cnt, d_scratch);                       \
    else k_quality_partials<M><<<g, 256, 0, s>>>(e, a, v, d_scratch);                          \
    k_quality_final<M><<<1, 1024, 0, s>>>(d_scratch, g, count, d_part3);
    switch (m) {
    case PARAPROX_MRE: PPX_QUALITY_CASE(PARAPROX_MRE) break;
    case PARAPROX_L2: PPX_QUALITY_CASE(PARAPROX_L2) break;
    default: PPX_QUALITY_CASE(PARAPROX_PSNR) break;
    }
#undef PPX_QUALITY_CASE
    count_launch(flat ? "quality_flat" : "quality_partials");
    count_launch("quality_final");
    return cudaGetLastError();
}

}  // namespace ppx
