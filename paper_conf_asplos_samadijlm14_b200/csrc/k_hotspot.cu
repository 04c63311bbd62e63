// k_hotspot.cu -- temporally blocked HotSpot steps (NEXT-4).
//
// HotSpot is a Stencil-Partition application (Table 1): the
// grid is partitioned into tiles that are advanced independently.  One CTA
// advances a tile by S <= 8 time steps from a single HBM read of T and P.
//
// Layout: a 48 x 128 or 96 x 128 box of cells (the tile plus an 8-cell halo on
// the accessed axes: 32 x 112 or 80 x 112 outputs for the exact stencil,
// 48 x 128 for the row scheme, which reads no neighbour row) is held in
// REGISTERS: warp w owns box rows 6w..6w+5 (12w..12w+11 in the tall box), lane l
// columns 4l..4l+3 of T; P (constant over the steps) in registers too, or in
// thread-private shared-memory slots in the tall box.  A step needs only
//  * the west / east neighbours: the adjacent lanes' edge columns (shuffles),
//  * the rows directly above / below a warp's rows: the neighbouring warps
//    publish their first and last rows in a ping-pong shared buffer (16 KB),
//    one barrier per step.
// The box edge has no neighbours: those cells turn to garbage one cell per
// step, which never reaches the outputs (8 halo cells >= S steps).  Clamp to
// the image edge (reading S7) is applied at read time in border tiles only:
// a cell on the first / last valid row or column reads itself in place of
// the missing neighbour, so out-of-image cells are never read by in-image
// ones and need no fix-up between steps.  The tall box (2 CTAs per SM instead
// of 3) computes 1.37 cells per output instead of 1.71: it is taken for steps
// with a row halo when it still gives every SM two tiles (8192^2 exact 47.1 ->
// 38.9 us per step; the paper's 1024^2 keeps the 48-row box).
//
// Each step adds the taps in the order of the tile kernels (rows ascending,
// columns ascending, fmaf from 0), then fmaf(alpha, P, .) + beta: bit-
// identical to S single steps.  The approximation shrinks the halo: the row
// scheme (rows {0}) stages no halo rows, needs no shared memory and no
// barrier; the column scheme (columns {0}) no shuffles.
//
// The first version staged T and P in shared memory with one dependent
// global load per staged row and thread and walked columns with a register
// window: 182 us per step at 8192^2, 1.5x slower than one plain pass per step.
#include "internal.h"

namespace ppx {

constexpr int kHsBW = 128, kHsWarps = 8, kHsMaxS = 8;
constexpr int kHsThreads = 32 * kHsWarps;
// box rows: 48 (6 per warp) or 96 (12 per warp: less halo overhead, 2 CTAs per
// SM instead of 3; the launch takes it when there are at least two tiles per SM
// and the step has a row halo)
template <int BH>
__host__ __device__ constexpr int hs_min_blocks() { return BH >= 96 ? 2 : 3; }

struct HsArgs {
    int n, h, w;
    int steps;
    const float* t;  // input temperature (rows 0..h-1 valid; no halos)
    const float* p;
    float* out;
    long long pitch, fs;  // shared layout of t, p, out
    float w9[3][3];       // folded taps at [a + 1][b + 1] (0 where not accessed)
    float alpha, beta;
    int tiles_x, tiles_y;
    int vec;  // 16-byte aligned rows everywhere: 128-bit loads and stores
    // optional peer halos (HotSpot row stripes): the ntop rows directly above
    // row 0 (T and P) and the nbot rows below row h-1, read from neighbour
    // buffers (CUDA IPC / NVLink); 0 rows = the image edge (clamp)
    const float *ptop_t, *ptop_p, *pbot_t, *pbot_p;
    int ntop, nbot;
    long long ppitch;
};

template <int HY, int HX, int BH>
struct HsGeom {
    static constexpr int RPW = BH / kHsWarps;           // box rows per warp
    static constexpr int OH = BH - 2 * kHsMaxS * HY;     // output rows per tile
    static constexpr int OW = kHsBW - 2 * kHsMaxS * HX;  // output columns per tile
    // P in registers (48-row box) or, for the 96-row box, in thread-private
    // shared slots ([row][thread] float4: conflict-free); then the ping-pong
    // of the warps' boundary rows
    static constexpr bool PREG = BH < 96;
    static constexpr int PBYTES = PREG ? 0 : RPW * kHsThreads * (int)sizeof(float4);
    static constexpr int SMEM = PBYTES + (HY ? 2 * kHsWarps * 2 * kHsBW * (int)sizeof(float) : 0);
};

__device__ __forceinline__ float hs_get(const float4& v, int c) {
    return c == 0 ? v.x : c == 1 ? v.y : c == 2 ? v.z : v.w;
}
__device__ __forceinline__ void hs_set(float4& v, int c, float x) {
    if (c == 0) v.x = x;
    else if (c == 1) v.y = x;
    else if (c == 2) v.z = x;
    else v.w = x;
}

// the S steps on the registers; EDGE: the box touches a valid-row or image-
// column edge (clamped neighbour reads), else the plain interior form
template <int HY, int HX, int RPW, bool EDGE, class PG>
__device__ __forceinline__ void hs_run(float4 (&T)[RPW], PG pget, const HsArgs& A,
                                       float* bnd, int wi, int lane, int oy, int ox, int lo, int hi) {
    const int S = A.steps;
    // per-row / per-column edge flags (EDGE only)
    bool top[RPW], bot[RPW], wst[4], est[4];
#pragma unroll
    for (int i = 0; i < RPW; ++i) {
        const int gy = oy + wi * RPW + i;
        top[i] = EDGE && gy == lo;
        bot[i] = EDGE && gy == hi;
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        const int gx = ox + 4 * lane + c;
        wst[c] = EDGE && gx == 0;
        est[c] = EDGE && gx == A.w - 1;
    }
    for (int k = 0; k < S; ++k) {
        float4 up = T[0], dn = T[RPW - 1];
        if constexpr (HY > 0) {
            float4* B = reinterpret_cast<float4*>(bnd + (k & 1) * (kHsWarps * 2 * kHsBW));
            B[(2 * wi) * (kHsBW / 4) + lane] = T[0];
            B[(2 * wi + 1) * (kHsBW / 4) + lane] = T[RPW - 1];
            __syncthreads();
            if (wi > 0) up = B[(2 * wi - 1) * (kHsBW / 4) + lane];
            if (wi < kHsWarps - 1) dn = B[(2 * wi + 2) * (kHsBW / 4) + lane];
        }
        float4 prev = up;  // old value of the row above
#pragma unroll
        for (int i = 0; i < RPW; ++i) {
            const float4 cur = T[i];
            const float4 nrt = (HY && top[i]) ? cur : prev;
            const float4 sth = (HY && bot[i]) ? cur : (i + 1 < RPW ? T[i + 1] : dn);
            float wl = 0.f, er = 0.f;
            if constexpr (HX > 0) {
                wl = __shfl_up_sync(0xffffffffu, cur.w, 1);
                er = __shfl_down_sync(0xffffffffu, cur.x, 1);
            }
            // the taps in order (N, W, C, E, S), column pairs (0,1) and (2,3)
            // in FFMA2 lanes where the operand pair is a register pair
            // (rows above / below, the centre, P); the west / east operands
            // straddle the pairs and take scalar FFMAs -- the same fp32 fma
            // per cell either way
            float2 a01 = make_float2(0.f, 0.f), a23 = make_float2(0.f, 0.f);
#pragma unroll
            for (int a = -HY; a <= HY; ++a)
#pragma unroll
                for (int b = -HX; b <= HX; ++b) {
                    if (a != 0 && b != 0) continue;
                    const float wt = A.w9[a + 1][b + 1];
                    if (b == 0) {
                        const float4 v = a < 0 ? nrt : (a > 0 ? sth : cur);
                        const float2 w2 = make_float2(wt, wt);
                        a01 = __ffma2_rn(w2, make_float2(v.x, v.y), a01);
                        a23 = __ffma2_rn(w2, make_float2(v.z, v.w), a23);
                    } else {
                        float v0, v1, v2, v3;  // the west (b < 0) or east neighbours
                        if (b < 0) {
                            v0 = wst[0] ? cur.x : wl;
                            v1 = wst[1] ? cur.y : cur.x;
                            v2 = wst[2] ? cur.z : cur.y;
                            v3 = wst[3] ? cur.w : cur.z;
                        } else {
                            v0 = est[0] ? cur.x : cur.y;
                            v1 = est[1] ? cur.y : cur.z;
                            v2 = est[2] ? cur.z : cur.w;
                            v3 = est[3] ? cur.w : er;
                        }
                        a01.x = __fmaf_rn(wt, v0, a01.x);
                        a01.y = __fmaf_rn(wt, v1, a01.y);
                        a23.x = __fmaf_rn(wt, v2, a23.x);
                        a23.y = __fmaf_rn(wt, v3, a23.y);
                    }
                }
            const float2 al2 = make_float2(A.alpha, A.alpha), be2 = make_float2(A.beta, A.beta);
            const float4 pv = pget(i);
            a01 = __fadd2_rn(__ffma2_rn(al2, make_float2(pv.x, pv.y), a01), be2);
            a23 = __fadd2_rn(__ffma2_rn(al2, make_float2(pv.z, pv.w), a23), be2);
            const float4 nv = make_float4(a01.x, a01.y, a23.x, a23.y);
            prev = cur;
            T[i] = nv;
        }
    }
}

template <int HY, int HX, int BH>
__global__ void __launch_bounds__(kHsThreads, hs_min_blocks<BH>()) k_hotspot_tb(const __grid_constant__ HsArgs A) {
    using G = HsGeom<HY, HX, BH>;
    constexpr int kHsRPW = G::RPW;
    extern __shared__ __align__(16) float smem_hs[];
    float4* Ps = reinterpret_cast<float4*>(smem_hs) + threadIdx.x;  // this thread's P slots, stride kHsThreads
    float* bnd = smem_hs + G::PBYTES / (int)sizeof(float);
    const int wi = threadIdx.x >> 5, lane = threadIdx.x & 31;
    int t = blockIdx.x;
    const int f = t / (A.tiles_x * A.tiles_y);
    t -= f * A.tiles_x * A.tiles_y;
    const int y0 = (t / A.tiles_x) * G::OH, x0 = (t % A.tiles_x) * G::OW;
    const int oy = y0 - kHsMaxS * HY, ox = x0 - kHsMaxS * HX;  // global coordinates of box cell (0, 0)
    const int lo = -A.ntop, hi = A.h - 1 + A.nbot;           // valid rows (peer halo rows included)
    const float* Tf = A.t + (long long)f * A.fs;
    const float* Pf = A.p + (long long)f * A.fs;

    // stage: the thread's 12 x 4 cells of T into registers (all loads in
    // flight at once) and of P into its shared slots (cp.async, no
    // registers); cells outside the valid rows / image columns read as 0
    // (never used by an in-image cell)
    float4 T[kHsRPW], Pv[G::PREG ? kHsRPW : 1];
    const int gx = ox + 4 * lane;
    const bool vec_ok = A.vec && gx >= 0 && gx + 3 < A.w;
#pragma unroll
    for (int i = 0; i < kHsRPW; ++i) {
        const int gy = oy + wi * kHsRPW + i;
        T[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        if constexpr (G::PREG) Pv[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        if (gy < lo || gy > hi) {
            if constexpr (!G::PREG) Ps[i * kHsThreads] = make_float4(0.f, 0.f, 0.f, 0.f);
            continue;
        }
        const float *ts, *ps;
        if (gy < 0) {
            const long long g = (long long)(A.ntop + gy) * A.ppitch;
            ts = A.ptop_t + g;
            ps = A.ptop_p + g;
        } else if (gy >= A.h) {
            const long long g = (long long)(gy - A.h) * A.ppitch;
            ts = A.pbot_t + g;
            ps = A.pbot_p + g;
        } else {
            const long long g = (long long)gy * A.pitch;
            ts = Tf + g;
            ps = Pf + g;
        }
        if (vec_ok) {
            T[i] = __ldcs(reinterpret_cast<const float4*>(ts + gx));
            if constexpr (G::PREG) {
                Pv[i] = __ldg(reinterpret_cast<const float4*>(ps + gx));
            } else {
                const uint32_t pdst = (uint32_t)__cvta_generic_to_shared(Ps + i * kHsThreads);
                asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(pdst), "l"(ps + gx) : "memory");
            }
        } else {
            float4 pv = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
            for (int c = 0; c < 4; ++c)
                if (gx + c >= 0 && gx + c < A.w) {
                    hs_set(T[i], c, ts[gx + c]);
                    hs_set(pv, c, ps[gx + c]);
                }
            if constexpr (G::PREG) Pv[i] = pv;
            else Ps[i * kHsThreads] = pv;
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
    asm volatile("cp.async.wait_group 0;" ::: "memory");  // own slots only: no barrier needed

    const bool edge = oy <= lo || oy + BH - 1 >= hi || ox <= 0 || ox + kHsBW - 1 >= A.w - 1;
    auto pget = [&](int i) -> float4 {
        if constexpr (G::PREG) return Pv[i];
        else return Ps[i * kHsThreads];
    };
    if (edge) hs_run<HY, HX, kHsRPW, true>(T, pget, A, bnd, wi, lane, oy, ox, lo, hi);
    else hs_run<HY, HX, kHsRPW, false>(T, pget, A, bnd, wi, lane, oy, ox, lo, hi);

    // the tile's outputs: box rows [8 HY, 8 HY + OH), columns [8 HX, 8 HX + OW)
    float* Of = A.out + (long long)f * A.fs;
#pragma unroll
    for (int i = 0; i < kHsRPW; ++i) {
        const int r = wi * kHsRPW + i;
        const int gy = oy + r;
        if (r < kHsMaxS * HY || r >= kHsMaxS * HY + G::OH || gy < 0 || gy >= A.h) continue;
        float* o = Of + (long long)gy * A.pitch;
        if (vec_ok && 4 * lane >= kHsMaxS * HX && 4 * lane + 3 < kHsMaxS * HX + G::OW) {
            __stcs(reinterpret_cast<float4*>(o + gx), T[i]);
        } else {
#pragma unroll
            for (int c = 0; c < 4; ++c) {
                const int bc = 4 * lane + c;
                if (bc >= kHsMaxS * HX && bc < kHsMaxS * HX + G::OW && gx + c >= 0 && gx + c < A.w)
                    __stcs(o + gx + c, hs_get(T[i], c));
            }
        }
    }
}

// taps of tap-index table order (rows, then columns ascending): the tile
// kernels add in this order, and so does k_hotspot_tb (zeros are exact)
cudaError_t launch_hotspot_tb(const Plan& p, const float* t, const float* pw, float* out, const View& v,
                              long long fs, float alpha, float beta, int steps, cudaStream_t s,
                              const HotspotPeer* peer) {
    if (steps < 1 || steps > kHsMaxS || p.separable || p.ky != 3 || p.kx != 3) return cudaErrorInvalidValue;
    for (int i = 0; i < p.ny; ++i)  // the kernel skips the corner taps: they must be zero
        for (int j = 0; j < p.nx; ++j)
            if (p.ay[i] != 0 && p.ax[j] != 0 && p.wf[i * p.nx + j] != 0.f) return cudaErrorInvalidValue;
    HsArgs A = {};
    A.n = v.n;
    A.h = v.h;
    A.w = v.w;
    A.steps = steps;
    A.t = t;
    A.p = pw;
    A.out = out;
    A.pitch = v.pitch;
    A.fs = fs;
    for (int i = 0; i < p.ny; ++i)
        for (int j = 0; j < p.nx; ++j) A.w9[p.ay[i] + 1][p.ax[j] + 1] = p.wf[i * p.nx + j];
    A.alpha = alpha;
    A.beta = beta;
    if (peer) {
        if (v.n != 1 || (peer->ntop && peer->ntop < steps * p.hy) || (peer->nbot && peer->nbot < steps * p.hy))
            return cudaErrorInvalidValue;  // the halo of `steps` steps must come from the peers
        A.ptop_t = peer->top_t;
        A.ptop_p = peer->top_p;
        A.pbot_t = peer->bot_t;
        A.pbot_p = peer->bot_p;
        A.ntop = peer->ntop;
        A.nbot = peer->nbot;
        A.ppitch = peer->pitch;
    }
    const auto al = [](const void* q) { return (reinterpret_cast<uintptr_t>(q) & 15) == 0; };
    A.vec = al(t) && al(pw) && al(out) && (v.pitch & 3) == 0 && (v.n == 1 || (fs & 3) == 0) &&
            (!peer || ((peer->pitch & 3) == 0 && al(peer->top_t) && al(peer->top_p) && al(peer->bot_t) &&
                       al(peer->bot_p)));
    int dev = 0, nsm = 0;  // the current device's SM count (a cheap attribute query)
    if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev) !=
                                                  cudaSuccess || nsm < 1)
        nsm = 148;
    auto tiles = [&](int oh, int ow) { return (long long)((v.h + oh - 1) / oh) * ((v.w + ow - 1) / ow) * v.n; };
    const int ow = p.hx ? HsGeom<0, 1, 48>::OW : HsGeom<0, 0, 48>::OW;
    const bool tall = p.hy && tiles(HsGeom<1, 0, 96>::OH, ow) >= 2LL * nsm;
    const int oh = !p.hy ? HsGeom<0, 0, 48>::OH : tall ? HsGeom<1, 0, 96>::OH : HsGeom<1, 0, 48>::OH;
    A.tiles_x = (v.w + ow - 1) / ow;
    A.tiles_y = (v.h + oh - 1) / oh;
    const long long nt = (long long)A.tiles_x * A.tiles_y * v.n;
    if (nt >= (1LL << 31)) return cudaErrorInvalidValue;
    auto launch = [&](auto kern, int smem) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        kern<<<(unsigned)nt, kHsThreads, smem, s>>>(A);
        return cudaGetLastError();
    };
    cudaError_t e;
    if (p.hy && p.hx) e = tall ? launch(k_hotspot_tb<1, 1, 96>, HsGeom<1, 1, 96>::SMEM)
                               : launch(k_hotspot_tb<1, 1, 48>, HsGeom<1, 1, 48>::SMEM);
    else if (p.hy) e = tall ? launch(k_hotspot_tb<1, 0, 96>, HsGeom<1, 0, 96>::SMEM)
                            : launch(k_hotspot_tb<1, 0, 48>, HsGeom<1, 0, 48>::SMEM);
    else if (p.hx) e = launch(k_hotspot_tb<0, 1, 48>, HsGeom<0, 1, 48>::SMEM);
    else e = launch(k_hotspot_tb<0, 0, 48>, HsGeom<0, 0, 48>::SMEM);
    if (e != cudaSuccess) return e;
    count_launch(p.hy && p.hx ? "hotspot_tb_f1_f1" : p.hy ? "hotspot_tb_f1_s0" : p.hx ? "hotspot_tb_s0_f1"
                                                                                        : "hotspot_tb_s0_s0");
    return cudaSuccess;
}

}  // namespace ppx

namespace ppx {

// cross-GPU step ordering for peer-halo passes: a single thread spins with
// acquire loads (system scope: the flag may live on a peer GPU) until the
// counter reaches `target`; the signal kernel publishes a counter with a
// release store after everything before it in the stream
__global__ void k_flag_wait(const volatile long long* flag, long long target) {
    long long v;
    for (;;) {
        asm volatile("ld.acquire.sys.global.b64 %0, [%1];" : "=l"(v) : "l"(flag) : "memory");
        if (v >= target) break;
        __nanosleep(200);
    }
}

__global__ void k_flag_set(long long* flag, long long value) {
    __threadfence_system();
    asm volatile("st.release.sys.global.b64 [%0], %1;" ::"l"(flag), "l"(value) : "memory");
}

cudaError_t launch_flag_wait(const long long* flag, long long target, cudaStream_t s) {
    k_flag_wait<<<1, 1, 0, s>>>(flag, target);
    count_launch("flag_wait");
    return cudaGetLastError();
}

cudaError_t launch_flag_set(long long* flag, long long value, cudaStream_t s) {
    k_flag_set<<<1, 1, 0, s>>>(flag, value);
    count_launch("flag_set");
    return cudaGetLastError();
}

}  // namespace ppx
