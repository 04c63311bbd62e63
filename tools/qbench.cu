// qbench.cu -- A/B of quality-reduction layouts (row a4: MRE / L2 partial sums
// of two fp32 images, 8 B of HBM read per pixel).  Standalone; not part of the
// library.  Uses the library's per-term arithmetic (quality.cuh) so only the
// work distribution differs between variants.
// Build: nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o qbench tools/qbench.cu
// Run on the GPU box: ./qbench [log2 floats per image] [nbuf]
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#include "../paper_conf_asplos_samadijlm14_b200/csrc/quality.cuh"

namespace ppx {
void count_launch(const char*) {}
}  // namespace ppx
using namespace ppx;

#define CK(x)                                                                          \
    do {                                                                               \
        cudaError_t e_ = (x);                                                          \
        if (e_ != cudaSuccess) {                                                       \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
            exit(1);                                                                   \
        }                                                                              \
    } while (0)

// V0/V3: persistent grid-stride, QU independent 128-bit loads of E and A in flight
template <int M, int QU, int MINB>
__global__ void __launch_bounds__(256, MINB) v_stride(const float* __restrict__ E, const float* __restrict__ A,
                                                      long long count, double* __restrict__ part) {
    QAcc<M> q;
    const long long n4 = count >> 2;
    const long long stride = (long long)gridDim.x * blockDim.x;
    const float4* e4 = reinterpret_cast<const float4*>(E);
    const float4* a4 = reinterpret_cast<const float4*>(A);
    for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += QU * stride) {
        float4 e[QU], a[QU];
#pragma unroll
        for (int u = 0; u < QU; ++u) {
            const long long j = i + u * stride;
            if (j < n4) {
                e[u] = __ldcs(e4 + j);
                a[u] = __ldcs(a4 + j);
            } else {
                e[u] = a[u] = make_float4(1.f, 1.f, 1.f, 1.f);
            }
        }
#pragma unroll
        for (int u = 0; u < QU; ++u) {
            if (i + u * stride >= n4) continue;
            q.add(e[u].x, a[u].x);
            q.add(e[u].y, a[u].y);
            q.add(e[u].z, a[u].z);
            q.add(e[u].w, a[u].w);
        }
    }
    double s0, s1;
    q.get(s0, s1);
    block_sum2(s0, s1);
    if (threadIdx.x == 0) {
        part[2 * blockIdx.x] = s0;
        part[2 * blockIdx.x + 1] = s1;
    }
}

// V1/V2: one CTA per contiguous chunk of 256 x QU float4 of each image; one
// partial pair per CTA.  LAST: the last CTA to finish (ticket) sums every
// partial in index order -- deterministic, one launch.
template <int M, int QU, bool LAST>
__global__ void __launch_bounds__(256) v_chunk(const float* __restrict__ E, const float* __restrict__ A,
                                               long long count, double* __restrict__ part,
                                               unsigned int* __restrict__ ticket, double* __restrict__ out2) {
    QAcc<M> q;
    const long long n4 = count >> 2;
    const long long base = (long long)blockIdx.x * (256 * QU) + threadIdx.x;
    const float4* e4 = reinterpret_cast<const float4*>(E);
    const float4* a4 = reinterpret_cast<const float4*>(A);
    float4 e[QU], a[QU];
#pragma unroll
    for (int u = 0; u < QU; ++u) {
        const long long j = base + u * 256;
        if (j < n4) {
            e[u] = __ldcs(e4 + j);
            a[u] = __ldcs(a4 + j);
        } else {
            e[u] = a[u] = make_float4(1.f, 1.f, 1.f, 1.f);
        }
    }
#pragma unroll
    for (int u = 0; u < QU; ++u) {
        if (base + u * 256 >= n4) continue;
        q.add(e[u].x, a[u].x);
        q.add(e[u].y, a[u].y);
        q.add(e[u].z, a[u].z);
        q.add(e[u].w, a[u].w);
    }
    double s0, s1;
    q.get(s0, s1);
    block_sum2(s0, s1);
    if (threadIdx.x == 0) {
        part[2 * blockIdx.x] = s0;
        part[2 * blockIdx.x + 1] = s1;
    }
    if constexpr (LAST) {
        __shared__ bool last;
        if (threadIdx.x == 0) {
            __threadfence();
            last = atomicAdd(ticket, 1u) == gridDim.x - 1;
        }
        __syncthreads();
        if (!last) return;
        __threadfence();
        double t0 = 0.0, t1 = 0.0;
        for (int k = threadIdx.x; k < (int)gridDim.x; k += blockDim.x) {
            t0 += __ldcg(part + 2 * k);
            t1 += __ldcg(part + 2 * k + 1);
        }
        block_sum2(t0, t1);
        if (threadIdx.x == 0) {
            out2[0] = t0;
            out2[1] = t1;
            *ticket = 0;
        }
    }
}

template <int M>
__global__ void __launch_bounds__(1024) k_final(const double* __restrict__ part, int g, double* __restrict__ out2) {
    double s0 = 0.0, s1 = 0.0;
    for (int k = threadIdx.x; k < g; k += blockDim.x) {
        s0 += part[2 * k];
        s1 += part[2 * k + 1];
    }
    block_sum2(s0, s1);
    if (threadIdx.x == 0) {
        out2[0] = s0;
        out2[1] = s1;
    }
}

int main(int argc, char** argv) {
    const int lg = argc > 1 ? atoi(argv[1]) : 24;
    const int nbuf = argc > 2 ? atoi(argv[2]) : 4;
    const long long n = 1ll << lg;
    int nsm = 0;
    CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
    std::vector<float*> E(nbuf), A(nbuf);
    std::vector<float> h(n);
    srand(1);
    for (long long i = 0; i < n; ++i) h[i] = 16.f + (float)(rand() % 220);
    for (int b = 0; b < nbuf; ++b) {
        CK(cudaMalloc(&E[b], n * 4));
        CK(cudaMalloc(&A[b], n * 4));
        CK(cudaMemcpy(E[b], h.data(), n * 4, cudaMemcpyHostToDevice));
        for (long long i = 0; i < n; ++i) h[i] += (float)((i * 7) % 5) - 2.f;
        CK(cudaMemcpy(A[b], h.data(), n * 4, cudaMemcpyHostToDevice));
    }
    double* part;
    double* out;
    unsigned int* ticket;
    const long long maxg = n / 1024 + 4096;
    CK(cudaMalloc(&part, maxg * 16));
    CK(cudaMalloc(&out, 64));
    CK(cudaMalloc(&ticket, 4));
    CK(cudaMemset(ticket, 0, 4));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    const int reps = 30;
    auto run = [&](const char* name, auto&& launch) {
        for (int k = 0; k < 3; ++k) launch(k % nbuf);
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e0));
        for (int k = 0; k < reps; ++k) launch(k % nbuf);
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        float ms;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        ms /= reps;
        double r[2];
        CK(cudaMemcpy(r, out, 16, cudaMemcpyDeviceToHost));
        printf("{\"variant\": \"%s\", \"floats\": %lld, \"us\": %.2f, \"gbs\": %.1f, \"s0\": %.17g, \"s1\": %.17g}\n",
               name, n, ms * 1e3, 8.0 * n / (ms * 1e-3) / 1e9, r[0], r[1]);
        fflush(stdout);
    };
#define VARIANTS(M, TAG)                                                                                       \
    run(TAG "_stride1184_qu4", [&](int b) {                                                                    \
        v_stride<M, 4, (M == PARAPROX_MRE ? 3 : 2)><<<1184, 256>>>(E[b], A[b], n, part);                       \
        k_final<M><<<1, 1024>>>(part, 1184, out);                                                              \
    });                                                                                                        \
    for (int occ : {2, 3, 4}) {                                                                                \
        char nm[64];                                                                                           \
        snprintf(nm, 64, TAG "_stride%dx%d_qu8", nsm, occ);                                                   \
        const int g = nsm * occ;                                                                               \
        run(nm, [&](int b) {                                                                                   \
            v_stride<M, 8, 2><<<g, 256>>>(E[b], A[b], n, part);                                                \
            k_final<M><<<1, 1024>>>(part, g, out);                                                             \
        });                                                                                                    \
    }                                                                                                          \
    run(TAG "_chunk_qu4_final", [&](int b) {                                                                   \
        const int g = (int)((n / 4 + 1023) / 1024);                                                            \
        v_chunk<M, 4, false><<<g, 256>>>(E[b], A[b], n, part, ticket, out);                                    \
        k_final<M><<<1, 1024>>>(part, g, out);                                                                 \
    });                                                                                                        \
    run(TAG "_chunk_qu4_last", [&](int b) {                                                                    \
        const int g = (int)((n / 4 + 1023) / 1024);                                                            \
        v_chunk<M, 4, true><<<g, 256>>>(E[b], A[b], n, part, ticket, out);                                     \
    });                                                                                                        \
    run(TAG "_chunk_qu8_last", [&](int b) {                                                                    \
        const int g = (int)((n / 4 + 2047) / 2048);                                                            \
        v_chunk<M, 8, true><<<g, 256>>>(E[b], A[b], n, part, ticket, out);                                     \
    });                                                                                                        \
    run(TAG "_chunk_qu2_last", [&](int b) {                                                                    \
        const int g = (int)((n / 4 + 511) / 512);                                                              \
        v_chunk<M, 2, true><<<g, 256>>>(E[b], A[b], n, part, ticket, out);                                     \
    });
    VARIANTS(PARAPROX_MRE, "mre")
    VARIANTS(PARAPROX_L2, "l2")
    return 0;
}
