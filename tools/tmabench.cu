// tmabench.cu -- A/B of TMA tile shapes for a streaming read+write of a
// 2-D fp32 image (the DRAM side of the stencil tile kernels): persistent CTAs
// load (bh x bw) boxes through a 4-D tensor map (8-float inner groups, so the
// box may be wider than TMA's 256-element limit), scale them, and write them
// back with 128-bit stores or a TMA store.  Standalone; not part of the library.
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o tmabench tools/tmabench.cu
//   ./tmabench [H] [W]
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>

#define CK(x)                                                                          \
    do {                                                                               \
        cudaError_t e_ = (x);                                                          \
        if (e_ != cudaSuccess) {                                                       \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
            exit(1);                                                                   \
        }                                                                              \
    } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

struct Args {
    float* out;
    const float* in;
    int H, W, bh, bw, tiles_x, ntiles, stages, tma_store;
    int stage_bytes;
    int map3d;      // 3-D map (inner dim = W) instead of 8-float groups
    int load_only;  // no stores: the TMA read ceiling
};

__global__ void __launch_bounds__(256) k_tiles_copy(const __grid_constant__ CUtensorMap in_map,
                                                    const __grid_constant__ CUtensorMap out_map, const Args A) {
    extern __shared__ __align__(128) unsigned char sm[];
    __shared__ uint64_t bar[8];
    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < A.stages; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    auto issue = [&](int t, int s) {
        const int ty = t / A.tiles_x, tx = t - ty * A.tiles_x;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(A.stage_bytes)
                     : "memory");
        if (A.map3d)
            asm volatile(
                "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
                "%4}], [%5];" ::"r"(su32(sm + s * A.stage_bytes)),
                "l"(&in_map), "r"(tx * A.bw), "r"(ty * A.bh), "r"(0), "r"(su32(&bar[s]))
                : "memory");
        else
            asm volatile(
                "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
                "%4, %5}], [%6];" ::"r"(su32(sm + s * A.stage_bytes)),
                "l"(&in_map), "r"(0), "r"(tx * A.bw / 8), "r"(ty * A.bh), "r"(0), "r"(su32(&bar[s]))
                : "memory");
    };
    if (tid == 0)
        for (int s = 0; s < A.stages - 1; ++s) {
            int t = blockIdx.x + s * gridDim.x;
            if (t < A.ntiles) issue(t, s);
        }
    int it = 0;
    for (int t = blockIdx.x; t < A.ntiles; t += gridDim.x, ++it) {
        const int s = it % A.stages;
        if (tid == 0) {
            int a = t + (A.stages - 1) * gridDim.x;
            if (a < A.ntiles) {
                if (A.tma_store) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
                issue(a, (it + A.stages - 1) % A.stages);
            }
        }
        uint32_t ok = 0;
        const uint32_t par = (it / A.stages) & 1;
        while (!ok)
            asm volatile(
                "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, "
                "p;\n\t}"
                : "=r"(ok)
                : "r"(su32(&bar[s])), "r"(par)
                : "memory");
        const int ty = t / A.tiles_x, tx = t - ty * A.tiles_x;
        float4* b = reinterpret_cast<float4*>(sm + s * A.stage_bytes);
        const int n4 = A.bh * A.bw / 4, w4 = A.bw / 4;
        if (A.load_only) {
            if (b[tid].x == 1.f) A.out[tid] = 1.f;  // never true (zeros): keeps the load
        } else if (A.tma_store) {
            for (int k = tid; k < n4; k += 256) {
                float4 v = b[k];
                b[k] = make_float4(0.5f * v.x, 0.5f * v.y, 0.5f * v.z, 0.5f * v.w);
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncthreads();
            if (tid == 0) {
                asm volatile(
                    "cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(&out_map),
                    "r"(su32(b)), "r"(0), "r"(tx * A.bw / 8), "r"(ty * A.bh), "r"(0)
                    : "memory");
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            }
        } else {
            for (int k = tid; k < n4; k += 256) {
                const int r = k / w4, c = k - r * w4;
                float4 v = b[k];
                __stcs(reinterpret_cast<float4*>(A.out + (long long)(ty * A.bh + r) * A.W + tx * A.bw) + c,
                       make_float4(0.5f * v.x, 0.5f * v.y, 0.5f * v.z, 0.5f * v.w));
            }
        }
        __syncthreads();
    }
    if (tid == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// cp.async (LDGSTS, 16 B per thread) ring instead of TMA
__global__ void __launch_bounds__(256) k_tiles_ldgsts(const Args A) {
    extern __shared__ __align__(128) unsigned char sm[];
    const int tid = threadIdx.x;
    const int n4 = A.bh * A.bw / 4, w4 = A.bw / 4;
    auto issue = [&](int t, int s) {
        const int ty = t / A.tiles_x, tx = t - ty * A.tiles_x;
        float4* b = reinterpret_cast<float4*>(sm + s * A.stage_bytes);
        for (int k = tid; k < n4; k += 256) {
            const int r = k / w4, c = k - r * w4;
            const float* g = A.in + (long long)(ty * A.bh + r) * A.W + tx * A.bw + 4 * c;
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(b + k)), "l"(g) : "memory");
        }
    };
    for (int s = 0; s < A.stages - 1; ++s) {
        int t = blockIdx.x + s * gridDim.x;
        if (t < A.ntiles) issue(t, s);
        asm volatile("cp.async.commit_group;" ::: "memory");
    }
    int it = 0;
    for (int t = blockIdx.x; t < A.ntiles; t += gridDim.x, ++it) {
        const int s = it % A.stages;
        int a = t + (A.stages - 1) * gridDim.x;
        if (a < A.ntiles) issue(a, (it + A.stages - 1) % A.stages);
        asm volatile("cp.async.commit_group;" ::: "memory");
        // groups committed after tile t's: stages - 1
        if (A.stages == 3) asm volatile("cp.async.wait_group 2;" ::: "memory");
        else if (A.stages == 4) asm volatile("cp.async.wait_group 3;" ::: "memory");
        else asm volatile("cp.async.wait_group 5;" ::: "memory");
        __syncthreads();
        const int ty = t / A.tiles_x, tx = t - ty * A.tiles_x;
        const float4* b = reinterpret_cast<const float4*>(sm + s * A.stage_bytes);
        for (int k = tid; k < n4; k += 256) {
            const int r = k / w4, c = k - r * w4;
            float4 v = b[k];
            __stcs(reinterpret_cast<float4*>(A.out + (long long)(ty * A.bh + r) * A.W + tx * A.bw) + c,
                   make_float4(0.5f * v.x, 0.5f * v.y, 0.5f * v.z, 0.5f * v.w));
        }
        __syncthreads();
    }
}

static PFN_cuTensorMapEncodeTiled_v12000 enc() {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q));
    return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
}

static void make_map3(CUtensorMap* m, float* base, int H, int W, int bh, int bw) {
    cuuint64_t dims[3] = {(cuuint64_t)W, (cuuint64_t)H, 1};
    cuuint64_t strides[2] = {(cuuint64_t)W * 4, (cuuint64_t)W * 4 * H};
    cuuint32_t box[3] = {(cuuint32_t)bw, (cuuint32_t)bh, 1};
    cuuint32_t es[3] = {1, 1, 1};
    CUresult r = enc()(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, base, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                       CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        fprintf(stderr, "encode3 failed %d\n", (int)r);
        exit(1);
    }
}

static void make_map(CUtensorMap* m, float* base, int H, int W, int bh, int bw) {
    cuuint64_t dims[4] = {8, (cuuint64_t)W / 8, (cuuint64_t)H, 1};
    cuuint64_t strides[3] = {32, (cuuint64_t)W * 4, (cuuint64_t)W * 4 * H};
    cuuint32_t box[4] = {8, (cuuint32_t)bw / 8, (cuuint32_t)bh, 1};
    cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = enc()(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, base, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                       CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
        fprintf(stderr, "encode failed %d (bh %d bw %d)\n", (int)r, bh, bw);
        exit(1);
    }
}

int main(int argc, char** argv) {
    const int H = argc > 1 ? atoi(argv[1]) : 32768, W = argc > 2 ? atoi(argv[2]) : 32768;
    const long long n = (long long)H * W;
    float *in, *out;
    CK(cudaMalloc(&in, n * 4));
    CK(cudaMalloc(&out, n * 4));
    CK(cudaMemset(in, 0, n * 4));
    int nsm;
    CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0));
    CK(cudaFuncSetAttribute(k_tiles_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    CK(cudaFuncSetAttribute(k_tiles_ldgsts, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
    auto timed = [&](auto&& run) {
        for (int k = 0; k < 3; ++k) run();
        CK(cudaDeviceSynchronize());
        CK(cudaEventRecord(e0));
        const int reps = 10;
        for (int k = 0; k < reps; ++k) run();
        CK(cudaEventRecord(e1));
        CK(cudaEventSynchronize(e1));
        CK(cudaGetLastError());
        float ms;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        return ms / reps;
    };
    const int shapes[][2] = {{64, 128}, {32, 256}, {8, 1024}};
    // mode: 0 TMA 4-D, 1 TMA 3-D, 2 LDGSTS; load_only for the TMA modes
    for (auto& sh : shapes)
        for (int mode : {0, 1, 2})
            for (int lo : {0, 1})
                for (int stages : {3, 4})
                    for (int per : {1, 2}) {
                        const int bh = sh[0], bw = sh[1];
                        const int sb = bh * bw * 4;
                        if ((long long)sb * stages * per > 210 * 1024) continue;
                        if (mode == 1 && bw > 256) continue;
                        if (mode == 2 && lo) continue;
                        CUtensorMap mi, mo;
                        if (mode == 1) {
                            make_map3(&mi, in, H, W, bh, bw);
                            make_map3(&mo, out, H, W, bh, bw);
                        } else {
                            make_map(&mi, in, H, W, bh, bw);
                            make_map(&mo, out, H, W, bh, bw);
                        }
                        Args A{out, in, H, W, bh, bw, W / bw, (H / bh) * (W / bw), stages, 0, sb, mode == 1, lo};
                        const int grid = nsm * per;
                        float ms = mode == 2 ? timed([&] { k_tiles_ldgsts<<<grid, 256, sb * stages>>>(A); })
                                             : timed([&] { k_tiles_copy<<<grid, 256, sb * stages>>>(mi, mo, A); });
                        printf("{\"mode\": %d, \"load_only\": %d, \"bh\": %d, \"bw\": %d, \"stages\": %d, \"ctas_per_sm\": %d, "
                               "\"us\": %.1f, \"gbs\": %.1f}\n",
                               mode, lo, bh, bw, stages, per, 1e3 * ms, (lo ? 4.0 : 8.0) * n / ms / 1e6);
                        fflush(stdout);
                    }
    return 0;
}
