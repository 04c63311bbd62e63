// k_quality.cu -- output-quality partial sums (Table 1
// metrics): mean relative error, L2-norm, PSNR.
//
// fp32 inputs, fp64 accumulation.  Deterministic: a fixed number of CTAs
// (kQualityBlocks, or fewer rows), each walking its rows in a fixed order,
// fixed warp-shuffle trees, then one CTA summing the per-CTA partials in a
// fixed order.  No atomics.  8 bytes of HBM read per pixel, nothing written.
#include "internal.h"

namespace ppx {

template <int M>
__device__ __forceinline__ void accum(float e, float a, double& s0, double& s1) {
    const double de = (double)e, da = (double)a;
    const double d = da - de;
    if (M == PARAPROX_MRE) {
        s0 += de != 0.0 ? fabs(d) / fabs(de) : (da == 0.0 ? 0.0 : 1.0);
    } else if (M == PARAPROX_L2) {
        s0 += d * d;
        s1 += de * de;
    } else {
        s0 += d * d;
    }
}

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

template <int M>
__global__ void __launch_bounds__(256) k_quality_partials(const float* __restrict__ E,
                                                          const float* __restrict__ A, View v,
                                                          double* __restrict__ part) {
    double s0 = 0.0, s1 = 0.0;
    const long long rows = (long long)v.n * v.h;
    const bool vec = ((v.pitch & 3) == 0) && ((v.fstride & 3) == 0) &&
                     ((((uintptr_t)E) | ((uintptr_t)A)) & 15) == 0;
    const int w4 = vec ? (v.w >> 2) : 0;
    for (long long R = blockIdx.x; R < rows; R += gridDim.x) {
        const long long f = R / v.h, y = R - f * v.h;
        const long long off = f * v.fstride + y * v.pitch;
        const float4* e4 = reinterpret_cast<const float4*>(E + off);
        const float4* a4 = reinterpret_cast<const float4*>(A + off);
        for (int x = threadIdx.x; x < w4; x += blockDim.x) {
            const float4 e = __ldcs(e4 + x), a = __ldcs(a4 + x);
            accum<M>(e.x, a.x, s0, s1);
            accum<M>(e.y, a.y, s0, s1);
            accum<M>(e.z, a.z, s0, s1);
            accum<M>(e.w, a.w, s0, s1);
        }
        for (int x = (w4 << 2) + threadIdx.x; x < v.w; x += blockDim.x)
            accum<M>(__ldcs(E + off + x), __ldcs(A + off + x), s0, s1);
    }
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
    const int g = (int)(rows < kQualityBlocks ? rows : kQualityBlocks);
    const double count = (double)v.n * (double)v.h * (double)v.w;
    switch (m) {
    case PARAPROX_MRE:
        k_quality_partials<PARAPROX_MRE><<<g, 256, 0, s>>>(e, a, v, d_scratch);
        k_quality_final<PARAPROX_MRE><<<1, 1024, 0, s>>>(d_scratch, g, count, d_part3);
        break;
    case PARAPROX_L2:
        k_quality_partials<PARAPROX_L2><<<g, 256, 0, s>>>(e, a, v, d_scratch);
        k_quality_final<PARAPROX_L2><<<1, 1024, 0, s>>>(d_scratch, g, count, d_part3);
        break;
    default:
        k_quality_partials<PARAPROX_PSNR><<<g, 256, 0, s>>>(e, a, v, d_scratch);
        k_quality_final<PARAPROX_PSNR><<<1, 1024, 0, s>>>(d_scratch, g, count, d_part3);
        break;
    }
    count_launch("quality_partials");
    count_launch("quality_final");
    return cudaGetLastError();
}

}  // namespace ppx
