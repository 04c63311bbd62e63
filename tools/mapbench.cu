// mapbench.cu -- A/B of streaming-map variants (out = w * in, fp32) for the
// centre-full-collapse kernel (k_pointwise_flat).  Standalone; not part of the
// library.  Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o mapbench tools/mapbench.cu
// Run on the GPU box: ./mapbench [log2 floats per buffer] [nbuf]
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>

#define CK(x)                                                                          \
    do {                                                                               \
        cudaError_t e_ = (x);                                                          \
        if (e_ != cudaSuccess) {                                                       \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
            exit(1);                                                                   \
        }                                                                              \
    } while (0)

// V0: the library's kernel: PU independent 128-bit evict-first loads, streaming stores
template <int PU, int HINT>
__global__ void __launch_bounds__(256) v_ldg(const float* __restrict__ in, float* __restrict__ out, long long count,
                                             float w) {
    const long long n4 = count >> 2;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const float4* i4 = reinterpret_cast<const float4*>(in);
    float4* o4 = reinterpret_cast<float4*>(out);
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += PU * stride) {
        float4 v[PU];
#pragma unroll
        for (int u = 0; u < PU; ++u)
            if (i + u * stride < n4) v[u] = HINT ? __ldcs(i4 + i + u * stride) : __ldg(i4 + i + u * stride);
#pragma unroll
        for (int u = 0; u < PU; ++u)
            if (i + u * stride < n4) {
                float4 r = make_float4(w * v[u].x, w * v[u].y, w * v[u].z, w * v[u].w);
                if (HINT) __stcs(o4 + i + u * stride, r);
                else o4[i + u * stride] = r;
            }
    }
}

// V1: 256-bit loads / stores (sm_100 .v8)
struct f8 {
    float v[8];
};
__device__ __forceinline__ f8 ld8(const float* p) {
    f8 r;
    asm volatile("ld.global.nc.L1::no_allocate.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3]), "=f"(r.v[4]), "=f"(r.v[5]), "=f"(r.v[6]),
                   "=f"(r.v[7])
                 : "l"(p));
    return r;
}
__device__ __forceinline__ void st8(float* p, const f8& r) {
    asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "f"(r.v[0]), "f"(r.v[1]), "f"(r.v[2]),
                 "f"(r.v[3]), "f"(r.v[4]), "f"(r.v[5]), "f"(r.v[6]), "f"(r.v[7])
                 : "memory");
}
template <int PU>
__global__ void __launch_bounds__(256) v_v8(const float* __restrict__ in, float* __restrict__ out, long long count,
                                            float w) {
    const long long n8 = count >> 3;
    const long long stride = (long long)gridDim.x * blockDim.x;
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n8; i += PU * stride) {
        f8 v[PU];
#pragma unroll
        for (int u = 0; u < PU; ++u)
            if (i + u * stride < n8) v[u] = ld8(in + 8 * (i + u * stride));
#pragma unroll
        for (int u = 0; u < PU; ++u)
            if (i + u * stride < n8) {
#pragma unroll
                for (int c = 0; c < 8; ++c) v[u].v[c] *= w;
                st8(out + 8 * (i + u * stride), v[u]);
            }
    }
}

// V2: non-persistent, torch-like: one block per 256 * PU float4
template <int PU>
__global__ void __launch_bounds__(256) v_blocks(const float* __restrict__ in, float* __restrict__ out, long long count,
                                                float w) {
    const long long n4 = count >> 2;
    const long long base = (long long)blockIdx.x * 256 * PU + threadIdx.x;
    const float4* i4 = reinterpret_cast<const float4*>(in);
    float4* o4 = reinterpret_cast<float4*>(out);
    float4 v[PU];
#pragma unroll
    for (int u = 0; u < PU; ++u)
        if (base + u * 256 < n4) v[u] = __ldg(i4 + base + u * 256);
#pragma unroll
    for (int u = 0; u < PU; ++u)
        if (base + u * 256 < n4) o4[base + u * 256] = make_float4(w * v[u].x, w * v[u].y, w * v[u].z, w * v[u].w);
}

// V3: TMA bulk ring: one producer thread issues cp.async.bulk global->smem,
// the CTA scales the chunk in place, one thread issues the bulk store back.
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
template <int CHUNK, int ST>
__global__ void __launch_bounds__(256) v_bulk(const float* __restrict__ in, float* __restrict__ out, long long count,
                                              float w) {
    extern __shared__ __align__(128) unsigned char sm[];
    __shared__ uint64_t bar[ST];
    const long long nchunks = (count * 4) / CHUNK;  // tail ignored in the A/B
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < ST; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](long long c, int s) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(CHUNK)
                     : "memory");
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                su32(sm + s * CHUNK)),
            "l"(in + c * (CHUNK / 4)), "r"(CHUNK), "r"(su32(&bar[s]))
            : "memory");
    };
    if (tid == 0)
        for (int s = 0; s < ST - 1; ++s) {
            long long c = blockIdx.x + (long long)s * gridDim.x;
            if (c < nchunks) issue(c, s);
        }
    int it = 0;
    for (long long c = blockIdx.x; c < nchunks; c += gridDim.x, ++it) {
        const int s = it % ST;
        if (tid == 0) {
            long long a = c + (long long)(ST - 1) * gridDim.x;
            if (a < nchunks) {
                // the stage being refilled was stored ST-1 iterations ago: wait for its read
                asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(ST - 2) : "memory");
                issue(a, (it + ST - 1) % ST);
            }
        }
        uint32_t ok = 0;
        const uint32_t par = (it / ST) & 1;
        while (!ok)
            asm volatile(
                "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, "
                "p;\n\t}"
                : "=r"(ok)
                : "r"(su32(&bar[s])), "r"(par)
                : "memory");
        float4* b = reinterpret_cast<float4*>(sm + s * CHUNK);
#pragma unroll
        for (int k = tid; k < CHUNK / 16; k += 256) {
            float4 v = b[k];
            b[k] = make_float4(w * v.x, w * v.y, w * v.z, w * v.w);
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        __syncthreads();
        if (tid == 0) {
            asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(out + c * (CHUNK / 4)),
                         "r"(su32(sm + s * CHUNK)), "r"(CHUNK)
                         : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        }
    }
    if (tid == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

template <class F>
float timeit(F&& f, int nbuf, int reps) {
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    for (int k = 0; k < 3; ++k) f(k % nbuf);
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(e0));
    for (int k = 0; k < reps; ++k) f(k % nbuf);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    CK(cudaGetLastError());
    return ms / reps;
}

int main(int argc, char** argv) {
    const int lg = argc > 1 ? atoi(argv[1]) : 30;
    const int nbuf = argc > 2 ? atoi(argv[2]) : 1;
    const int reps = argc > 3 ? atoi(argv[3]) : 20;
    const long long count = 1ll << lg;
    int nsm;
    CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
    std::vector<float*> ins(nbuf), outs(nbuf);
    for (int k = 0; k < nbuf; ++k) {
        CK(cudaMalloc(&ins[k], count * 4));
        CK(cudaMalloc(&outs[k], count * 4));
        CK(cudaMemset(ins[k], 0, count * 4));
    }
    const double bytes = 8.0 * count;
    auto rep = [&](const char* name, float ms) {
        printf("{\"lg\": %d, \"nbuf\": %d, \"variant\": \"%s\", \"us\": %.2f, \"gbs\": %.1f}\n", lg, nbuf, name,
               1e3 * ms, bytes / ms / 1e6);
        fflush(stdout);
    };
    rep("memcpy_d2d", timeit([&](int k) { CK(cudaMemcpyAsync(outs[k], ins[k], count * 4, cudaMemcpyDeviceToDevice)); },
                             nbuf, reps));
    const float w = 0.5f;
#define LDG(PU, H, MUL)                                                                                 \
    rep("ldg_pu" #PU "_h" #H "_x" #MUL,                                                                  \
        timeit([&](int k) { v_ldg<PU, H><<<nsm * MUL, 256>>>(ins[k], outs[k], count, w); }, nbuf, reps));
    LDG(8, 1, 8) LDG(8, 0, 8) LDG(4, 1, 8) LDG(4, 0, 8) LDG(16, 1, 8) LDG(8, 1, 4) LDG(4, 0, 16) LDG(2, 0, 8)
        LDG(8, 1, 16)
#define V8(PU, MUL) \
    rep("v8_pu" #PU "_x" #MUL, timeit([&](int k) { v_v8<PU><<<nsm * MUL, 256>>>(ins[k], outs[k], count, w); }, nbuf, reps));
            V8(4, 8) V8(2, 8) V8(8, 8) V8(4, 4)
#define BLK(PU)                                                                                              \
    rep("blocks_pu" #PU, timeit([&](int k) {                                                               \
            v_blocks<PU><<<(unsigned)((count / 4 + 256 * PU - 1) / (256 * PU)), 256>>>(ins[k], outs[k], count, w); \
        }, nbuf, reps));
                BLK(4) BLK(8) BLK(2)
#define BULK(CH, ST, PER)                                                                                   \
    {                                                                                                       \
        auto kf = v_bulk<CH, ST>;                                                                           \
        CK(cudaFuncSetAttribute(kf, cudaFuncAttributeMaxDynamicSharedMemorySize, CH * ST));                 \
        rep("bulk_" #CH "_st" #ST "_per" #PER,                                                              \
            timeit([&](int k) { kf<<<nsm * PER, 256, CH * ST>>>(ins[k], outs[k], count, w); }, nbuf, reps)); \
    }
                    BULK(16384, 4, 2) BULK(16384, 6, 2) BULK(32768, 3, 2) BULK(32768, 6, 1) BULK(8192, 8, 2)
                        BULK(16384, 4, 3) BULK(65536, 3, 1)
    return 0;
}
