// k_pointwise.cu -- plans whose accessed offsets are only (0, 0).
//
// At full reach the centre scheme lets the tile centre stand in for every
// neighbour ("the center element ... approximates all neighboring values",
// PAPER.md L1158-1162 Fig. 6a): the folded filter is one tap w' = sum of all
// weights, so the stencil degenerates to the map out = w' * in -- no halo, no
// neighbour, nothing to stage.  This kernel streams it at copy speed: each
// CTA streams one contiguous chunk, kPU = 4 independent 128-bit loads in
// flight per thread (evict-first), 128-bit streaming stores.  8 B of HBM per pixel.
//
// Rounding matches the tile kernels bit for bit: dense fmaf(w, x, 0);
// separable fmaf(wy, fmaf(wx, x, 0), 0) (horizontal, then vertical pass).
#include <algorithm>
#include <cmath>

#include "quality.cuh"

namespace ppx {

constexpr int kPU = 4;  // float4 loads in flight per thread
static_assert(kPU >= 4, "quality_scratch_doubles() sizes one partial pair per 4096 floats");

// streaming 128-bit load, evict-first
__device__ __forceinline__ float4 ld_stream(const float4* p) { return __ldcs(p); }

template <bool SEP>
__device__ __forceinline__ float pw(float x, float w0, float w1) {
    if constexpr (SEP) return __fmaf_rn(w0, __fmaf_rn(w1, x, 0.f), 0.f);
    else return __fmaf_rn(w0, x, 0.f);
}

template <bool SEP>
__device__ __forceinline__ float4 pw4(float4 x, float w0, float w1) {
    return make_float4(pw<SEP>(x.x, w0, w1), pw<SEP>(x.y, w0, w1), pw<SEP>(x.z, w0, w1), pw<SEP>(x.w, w0, w1));
}

__device__ __forceinline__ float plus(float r, float a, const Addend& add) {
    return __fadd_rn(__fmaf_rn(add.alpha, a, r), add.beta);
}
__device__ __forceinline__ float4 plus4(float4 r, float4 a, const Addend& add) {
    return make_float4(plus(r.x, a.x, add), plus(r.y, a.y, add), plus(r.z, a.z, add), plus(r.w, a.w, add));
}
// a centre-only plan has no neighbours, so consecutive steps of an iterated
// map (HotSpot at full collapse) fuse: the value stays in a register, each
// step rounded exactly as a separate launch would round it
template <bool SEP>
__device__ __forceinline__ float4 steps4(float4 x, float4 a, float w0, float w1, const Addend& add) {
    for (int k = 0; k < add.steps; ++k) x = plus4(pw4<SEP>(x, w0, w1), a, add);
    return x;
}
template <bool SEP>
__device__ __forceinline__ float steps1(float x, float a, float w0, float w1, const Addend& add) {
    for (int k = 0; k < add.steps; ++k) x = plus(pw<SEP>(x, w0, w1), a, add);
    return x;
}

// contiguous input and output, 16-byte aligned: one flat array.  One CTA per
// contiguous chunk of 256 x kPU float4 (not a persistent grid-stride loop):
// the requests in flight at any time then cover one contiguous window of the
// array, which the A/B in tools/mapbench.cu measured 13-16 % faster at 4 GiB
// (6.9 TB/s, above cudaMemcpy's 6.66) than the grid-stride form, whose kPU
// loads per thread land a whole grid stride (4.8 MB) apart.
template <bool SEP, int PU = kPU>
__global__ void __launch_bounds__(256) k_pointwise_flat(const float* __restrict__ in, float* __restrict__ out,
                                                        long long count, float w0, float w1, const Addend add) {
    const long long n4 = count >> 2;
    const long long base = (long long)blockIdx.x * (256 * PU) + threadIdx.x;
    const float4* i4 = reinterpret_cast<const float4*>(in);
    float4* o4 = reinterpret_cast<float4*>(out);
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    float4 v[PU];
#pragma unroll
    for (int u = 0; u < PU; ++u)
        if (base + u * 256 < n4) v[u] = ld_stream(i4 + base + u * 256);
#pragma unroll
    for (int u = 0; u < PU; ++u)
        if (base + u * 256 < n4) {
            const long long i = base + u * 256;
            const float4 r = add.p ? steps4<SEP>(v[u], __ldcs(reinterpret_cast<const float4*>(add.p) + i), w0, w1, add)
                                   : pw4<SEP>(v[u], w0, w1);
            __stcs(o4 + i, r);
        }
    if (blockIdx.x == gridDim.x - 1)
        for (long long x = (n4 << 2) + threadIdx.x; x < count; x += blockDim.x)
            out[x] = add.p ? steps1<SEP>(in[x], add.p[x], w0, w1, add) : pw<SEP>(in[x], w0, w1);
}

// fused quality (the tuner's centre candidates): compare w' x with the
// reference instead of storing; one CTA per contiguous chunk of 256 x kPU
// float4 (the map kernel's layout), 2 fp64 partials per CTA, deterministic
template <bool SEP>
__global__ void __launch_bounds__(256) k_pointwise_flat_q(const float* __restrict__ in, const float* __restrict__ ref,
                                                          long long count, float w0, float w1, int metric,
                                                          int ref_exact, double* __restrict__ part) {
    const long long n4 = count >> 2;
    const long long base = (long long)blockIdx.x * (256 * kPU) + threadIdx.x;
    const float4* i4 = reinterpret_cast<const float4*>(in);
    const float4* r4 = reinterpret_cast<const float4*>(ref);
    RAcc q;
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    auto term = [&](float v, float r) { q.add(metric, ref_exact ? r : v, ref_exact ? v : r); };
    float4 v[kPU], r[kPU];
#pragma unroll
    for (int u = 0; u < kPU; ++u)
        if (base + u * 256 < n4) {
            v[u] = ld_stream(i4 + base + u * 256);
            r[u] = __ldcs(r4 + base + u * 256);
        }
#pragma unroll
    for (int u = 0; u < kPU; ++u)
        if (base + u * 256 < n4) {
            const float4 a = pw4<SEP>(v[u], w0, w1);
            term(a.x, r[u].x);
            term(a.y, r[u].y);
            term(a.z, r[u].z);
            term(a.w, r[u].w);
        }
    if (blockIdx.x == gridDim.x - 1)
        for (long long x = (n4 << 2) + threadIdx.x; x < count; x += blockDim.x) term(pw<SEP>(in[x], w0, w1), ref[x]);
    double s0, s1;
    q.get(metric, s0, s1);
    block_sum2(s0, s1);
    if (threadIdx.x == 0) {
        part[2 * blockIdx.x] = s0;
        part[2 * blockIdx.x + 1] = s1;
    }
}

// any layout: rows of the output image, 128-bit where both rows allow it
template <bool SEP>
__global__ void __launch_bounds__(256) k_pointwise_rows(const float* __restrict__ in, View v,
                                                        float* __restrict__ out, long long opitch,
                                                        long long ofs, float w0, float w1, const Addend add) {
    const long long rows = (long long)v.n * v.h;
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    for (long long R = blockIdx.x; R < rows; R += gridDim.x) {  // grid = rows unless > 2^31-1
        const long long f = R / v.h, y = R - f * v.h;
        const float* src = in + f * v.fstride + y * v.pitch;
        float* dst = out + f * ofs + y * opitch;
        const float* ap = add.p ? add.p + f * add.fstride + y * add.pitch : nullptr;
        const bool vec = ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst) |
                           reinterpret_cast<uintptr_t>(ap)) & 15) == 0;
        const int w4 = vec ? (v.w >> 2) : 0;
        for (int x = threadIdx.x; x < w4; x += blockDim.x) {
            const float4 xv = __ldcs(reinterpret_cast<const float4*>(src) + x);
            const float4 r = ap ? steps4<SEP>(xv, __ldcs(reinterpret_cast<const float4*>(ap) + x), w0, w1, add)
                                : pw4<SEP>(xv, w0, w1);
            __stcs(reinterpret_cast<float4*>(dst) + x, r);
        }
        for (int x = (w4 << 2) + threadIdx.x; x < v.w; x += blockDim.x) {
            const float r = ap ? steps1<SEP>(__ldcs(src + x), __ldcs(ap + x), w0, w1, add) : pw<SEP>(__ldcs(src + x), w0, w1);
            __stcs(dst + x, r);
        }
    }
}

cudaError_t launch_pointwise(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                             long long ofs, cudaStream_t s, const Addend* addp) {
    const Addend add = addp ? *addp : Addend();
    cudaError_t err = cudaSuccess;
    const float w0 = p.separable ? p.wyf[0] : p.wf[0];
    const float w1 = p.separable ? p.wxf[0] : 1.f;
    const long long count = (long long)v.n * v.h * v.w;
    const bool flat = v.pitch == v.w && opitch == v.w && (v.n == 1 || (v.fstride == (long long)v.h * v.w &&
                      ofs == (long long)v.h * v.w)) &&
                      (((reinterpret_cast<uintptr_t>(in) | reinterpret_cast<uintptr_t>(out)) & 15) == 0) &&
                      (!add.p || (add.pitch == v.w && (v.n == 1 || add.fstride == (long long)v.h * v.w) &&
                                  (reinterpret_cast<uintptr_t>(add.p) & 15) == 0));
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(256);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    if (flat) {
        // float4 per thread: kPU (16 KiB per CTA), or fewer when that leaves a
        // mostly empty last wave of CTAs (c2: 4096 CTAs = 3.5 waves of the
        // 1184 resident; 8 KiB chunks make 6.9 waves)
        int pu = kPU;
        {
            static int resident = 0;  // CTAs per GPU (SMs x 8 at 256 threads)
            if (!resident) {
                int dev = 0, sms = 148, occ = 8;
                if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
                cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_pointwise_flat<false>, 256, 0);
                resident = sms * std::max(1, occ);
            }
            double best = 0.0;
            for (int c : {kPU, 2, 1}) {
                const double waves = (double)((count / 4 + 256LL * c - 1) / (256LL * c)) / resident;
                const double eff = waves / std::ceil(waves);
                if (eff > best + 0.02) {
                    best = eff;
                    pu = c;
                }
            }
        }
        const long long per = 256LL * pu;
        const long long want = (count / 4 + per - 1) / per;
        cfg.gridDim = dim3((unsigned)std::max<long long>(1, std::min<long long>(want, 0x7fffffffLL)));
#define PPX_MAP_LAUNCH(PU)                                                                                  \
    err = p.separable ? cudaLaunchKernelEx(&cfg, k_pointwise_flat<true, PU>, in, out, count, w0, w1, add)   \
                      : cudaLaunchKernelEx(&cfg, k_pointwise_flat<false, PU>, in, out, count, w0, w1, add);
        if (pu == 1) {
            PPX_MAP_LAUNCH(1)
        } else if (pu == 2) {
            PPX_MAP_LAUNCH(2)
        } else {
            PPX_MAP_LAUNCH(kPU)
        }
#undef PPX_MAP_LAUNCH
        count_launch(p.separable ? "sep_map" : "dense_map");
    } else {
        const long long rows = (long long)v.n * v.h;
        cfg.gridDim = dim3((unsigned)std::min<long long>(rows, 0x7fffffffLL));
        err = p.separable ? cudaLaunchKernelEx(&cfg, k_pointwise_rows<true>, in, v, out, opitch, ofs, w0, w1, add)
                          : cudaLaunchKernelEx(&cfg, k_pointwise_rows<false>, in, v, out, opitch, ofs, w0, w1, add);
        count_launch(p.separable ? "sep_map_rows" : "dense_map_rows");
    }
    if (err != cudaSuccess) return err;
    return cudaGetLastError();
}

}  // namespace ppx

namespace ppx {

// the map kernel in fused-quality mode; false when the layout is not flat
bool launch_pointwise_quality(const Plan& p, const float* in, const View& v, const float* ref, long long rpitch,
                              long long rfs, int metric, int ref_exact, double* part, int* grid_out, cudaStream_t s,
                              cudaError_t* err) {
    const long long count = (long long)v.n * v.h * v.w;
    const bool flat = v.pitch == v.w && rpitch == v.w && (v.n == 1 || (v.fstride == (long long)v.h * v.w &&
                      rfs == (long long)v.h * v.w)) && v.lo == 0 &&
                      (((reinterpret_cast<uintptr_t>(in) | reinterpret_cast<uintptr_t>(ref)) & 15) == 0);
    if (!flat) return false;
    const float w0 = p.separable ? p.wyf[0] : p.wf[0];
    const float w1 = p.separable ? p.wxf[0] : 1.f;
    // one CTA per 256 x kPU float4 (<= quality_scratch_doubles(count) / 2 partial pairs)
    const long long grid = std::max<long long>(1, (count / 4 + 256 * kPU - 1) / (256 * kPU));
    if (grid >= (1LL << 31)) {
        *err = cudaErrorInvalidValue;
        return true;
    }
    if (p.separable)
        k_pointwise_flat_q<true><<<(unsigned)grid, 256, 0, s>>>(in, ref, count, w0, w1, metric, ref_exact, part);
    else
        k_pointwise_flat_q<false><<<(unsigned)grid, 256, 0, s>>>(in, ref, count, w0, w1, metric, ref_exact, part);
    count_launch(p.separable ? "sep_map_quality" : "dense_map_quality");
    *grid_out = (int)grid;
    *err = cudaGetLastError();
    return true;
}

}  // namespace ppx
