// k_quality.cu -- output-quality partial sums (Table 1
// metrics): mean relative error, L2-norm, PSNR.
//
// fp32 inputs; fp64 per-thread sums (MRE terms formed as fp32 pairs), fp64
// reductions.  Deterministic: a fixed number of CTAs
// (kQualityBlocks, or fewer rows), each walking its rows in a fixed order,
// fixed warp-shuffle trees, then one CTA summing the per-CTA partials in a
// fixed order.  No atomics.  8 bytes of HBM read per pixel, nothing written.
#include "quality.cuh"

namespace ppx {

// Programmatic dependent launch: every quality kernel is launched with
// programmatic stream serialisation, so its CTAs may be scheduled while the
// previous kernel on the stream (a stencil, or the previous reduction level)
// drains.  griddepcontrol.wait blocks until that kernel has completed and its
// writes are visible; launch_dependents then lets the next level be scheduled
// early in turn.  Both are no-ops for a plain launch.
__device__ __forceinline__ void pdl_wait_and_release() {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

template <typename... KArgs, typename... Args>
static cudaError_t launch_pdl(void (*k)(KArgs...), int grid, int block, cudaStream_t s, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(block);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

// Contiguous images (pitch == w, frames back to back) are one flat array:
// one CTA per contiguous chunk of 256 x kQU float4 of E and of A (all loads of
// a thread issued before any arithmetic), one partial pair per CTA.  The
// requests in flight then cover one contiguous window of both arrays, as in
// the map kernel; tools/qbench.cu measured this 13-18 % faster at 64 MiB per
// image than the persistent grid-stride loop it replaced (equal at 1 GiB).
// Other layouts walk rows.
constexpr int kQU = 4;  // float4 loads of each image in flight per thread
constexpr long long kQChunk = 256LL * kQU * 4;  // floats of each image per CTA
static_assert(kQU >= 4, "quality_scratch_doubles() sizes one partial pair per 4096 floats");

template <int M>
__global__ void __launch_bounds__(256) k_quality_flat(const float* __restrict__ E, const float* __restrict__ A,
                                                      long long count, double* __restrict__ part) {
    pdl_wait_and_release();
    QAcc<M> q;
    const long long n4 = count >> 2;
    const long long base = (long long)blockIdx.x * (256 * kQU) + threadIdx.x;
    const float4* e4 = reinterpret_cast<const float4*>(E);
    const float4* a4 = reinterpret_cast<const float4*>(A);
    auto sweep = [&](auto&& op) {
        float4 e[kQU], a[kQU];
#pragma unroll
        for (int u = 0; u < kQU; ++u) {
            const long long j = base + u * 256;
            if (j < n4) {
                e[u] = __ldcs(e4 + j);
                a[u] = __ldcs(a4 + j);
            } else {
                e[u] = a[u] = make_float4(1.f, 1.f, 1.f, 1.f);  // |1-1|/|1| = 0, (1-1)^2 = 0
            }
        }
#pragma unroll
        for (int u = 0; u < kQU; ++u) {
            if (base + u * 256 >= n4) continue;  // (L2 would count the padding's E^2)
            op(e[u].x, a[u].x);
            op(e[u].y, a[u].y);
            op(e[u].z, a[u].z);
            op(e[u].w, a[u].w);
        }
        if (blockIdx.x == gridDim.x - 1)
            for (long long x = (n4 << 2) + threadIdx.x; x < count; x += blockDim.x) op(E[x], A[x]);
    };
    sweep([&](float e, float a) { q.add(e, a); });
    if constexpr (M == PARAPROX_MRE)
        if (__syncthreads_or(q.bad)) {
            q.reset();
            sweep([&](float e, float a) { q.fix(e, a); });
        }
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
    pdl_wait_and_release();
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
        if (__syncthreads_or(q.bad)) {
            q.reset();
            sweep([&](float e, float a) { q.fix(e, a); });
        }
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
    pdl_wait_and_release();
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

// d_scratch: >= quality_scratch_doubles(n * h * w) doubles.  Writes 3 doubles at d_part3.
cudaError_t launch_quality(const float* e, const float* a, const View& v, paraprox_metric m,
                           double* d_part3, double* d_scratch, cudaStream_t s) {
    const long long rows = (long long)v.n * v.h;
    const double count = (double)v.n * (double)v.h * (double)v.w;
    const bool flat = v.pitch == v.w && (v.n == 1 || v.fstride == (long long)v.h * v.w) &&
                      ((((uintptr_t)e) | ((uintptr_t)a)) & 15) == 0;
    const long long cnt = (long long)v.n * v.h * v.w;
    int g;
    if (flat) {
        const long long chunks = (cnt + kQChunk - 1) / kQChunk;
        if (chunks >= (1LL << 31)) return cudaErrorInvalidValue;
        g = (int)(chunks > 0 ? chunks : 1);
    } else {
        g = (int)(rows < kQualityBlocks ? rows : kQualityBlocks);
    }
    cudaError_t err;
#define PPX_QUALITY_CASE(M)                                                                    \
    if (flat) err = launch_pdl(k_quality_flat<M>, g, 256, s, e, a, cnt, d_scratch);            \
    else err = launch_pdl(k_quality_partials<M>, g, 256, s, e, a, v, d_scratch);
    switch (m) {
    case PARAPROX_MRE: PPX_QUALITY_CASE(PARAPROX_MRE) break;
    case PARAPROX_L2: PPX_QUALITY_CASE(PARAPROX_L2) break;
    default: PPX_QUALITY_CASE(PARAPROX_PSNR) break;
    }
#undef PPX_QUALITY_CASE
    if (err != cudaSuccess) return err;
    count_launch(flat ? "quality_flat" : "quality_partials");
    return launch_quality_final(d_scratch, g, count, m, d_part3, s);
}

// level 2 of the partial-pair reduction: CTA b sums pairs [b kFold, (b+1) kFold)
// in a fixed tree (a single final CTA would read 41 k pairs at c2's tuner size
// in ~22 us, 262 k at c4)
constexpr int kFold = 2048;
__global__ void __launch_bounds__(256) k_quality_fold(const double* __restrict__ part, int g,
                                                      double* __restrict__ out) {
    pdl_wait_and_release();
    double s0 = 0.0, s1 = 0.0;
    const int k0 = blockIdx.x * kFold;
    const int k1 = min(g, k0 + kFold);
    for (int k = k0 + threadIdx.x; k < k1; k += blockDim.x) {
        s0 += part[2 * k];
        s1 += part[2 * k + 1];
    }
    block_sum2(s0, s1);
    if (threadIdx.x == 0) {
        out[2 * blockIdx.x] = s0;
        out[2 * blockIdx.x + 1] = s1;
    }
}

// sums g partial pairs at d_scratch (fixed order; above 4096 pairs via one
// fold level written behind them, see quality_scratch_doubles) into d_part3
cudaError_t launch_quality_final(const double* d_scratch, int g, double count, paraprox_metric m, double* d_part3,
                                 cudaStream_t s) {
    if (g > 2 * kFold) {
        double* lvl2 = const_cast<double*>(d_scratch) + 2 * (size_t)g;
        const int g2 = (g + kFold - 1) / kFold;
        cudaError_t err = launch_pdl(k_quality_fold, g2, 256, s, d_scratch, g, lvl2);
        if (err != cudaSuccess) return err;
        count_launch("quality_fold");
        d_scratch = lvl2;
        g = g2;
    }
    cudaError_t err;
    switch (m) {
    case PARAPROX_MRE: err = launch_pdl(k_quality_final<PARAPROX_MRE>, 1, 1024, s, d_scratch, g, count, d_part3); break;
    case PARAPROX_L2: err = launch_pdl(k_quality_final<PARAPROX_L2>, 1, 1024, s, d_scratch, g, count, d_part3); break;
    default: err = launch_pdl(k_quality_final<PARAPROX_PSNR>, 1, 1024, s, d_scratch, g, count, d_part3); break;
    }
    if (err != cudaSuccess) return err;
    count_launch("quality_final");
    return cudaGetLastError();
}

size_t quality_scratch_pairs(long long count) {
    const long long chunks = (count + 4095) / 4096;
    return (size_t)(chunks > kQualityBlocks ? chunks : kQualityBlocks);
}

size_t quality_scratch_doubles(long long count) {
    const size_t g = quality_scratch_pairs(count);
    return 2 * g + 2 * (g / kFold + 1);  // partial pairs + the fold level
}

}  // namespace ppx
