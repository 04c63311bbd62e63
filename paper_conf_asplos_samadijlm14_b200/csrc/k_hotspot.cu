// k_hotspot.cu -- temporally blocked HotSpot steps (NEXT-4).
//
// HotSpot is a Stencil-Partition application (Table 1): the
// grid is partitioned into tiles that are advanced independently.  Here one
// CTA advances a 32 x 128 output tile by S <= 8 time steps from a single HBM
// read: it stages T and P with an S-cell halo (clamped at the image edges) in
// shared memory and computes step k over the tile grown by (S - k) cells of
// halo, ping-ponging two shared buffers; cells outside the image are reset to
// their clamped in-image cell after every step, so every step sees exactly the
// clamp-to-edge borders of a single step (reading S7).  HBM traffic: 12 bytes
// per output pixel per S steps instead of per step.
//
// The approximation shrinks the halo: the folded 3x3 plan's accessed offsets
// (row scheme: rows {0}; column: columns {0}) set HY / HX, so the row scheme
// stages no halo rows at all.  Each step adds the taps in the order of the
// tile kernels (rows ascending, columns ascending, fmaf from 0), then
// fmaf(alpha, P, .) + beta: bit-identical to S single steps.
#include "internal.h"

namespace ppx {

constexpr int kHsTH = 32, kHsTW = 128, kHsMaxS = 8;

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
    // optional peer halos (HotSpot row stripes): the ntop rows directly above
    // row 0 (T and P) and the nbot rows below row h-1, read from neighbour
    // buffers (CUDA IPC / NVLink); 0 rows = the image edge (clamp)
    const float *ptop_t, *ptop_p, *pbot_t, *pbot_p;
    int ntop, nbot;
    long long ppitch;
};

template <int HY, int HX>
struct HsGeom {
    static constexpr int RH = kHsTH + 2 * kHsMaxS * HY;  // staged rows (max halo)
    static constexpr int RW = kHsTW + 2 * kHsMaxS * HX;  // staged columns = threads per row group
    static constexpr int THREADS = 2 * RW;               // two row groups
    static constexpr int SMEM = 3 * RH * RW * (int)sizeof(float);
};

// Each thread owns one column of the step's region and half of its rows, and
// walks down them with a 3 x (2HX+1) register window: 2HX+1 shared loads of
// T, one of P and one store per cell and step.
template <int HY, int HX>
__global__ void __launch_bounds__(HsGeom<HY, HX>::THREADS, 2) k_hotspot_tb(const __grid_constant__ HsArgs A) {
    using G = HsGeom<HY, HX>;
    constexpr int RW = G::RW;
    extern __shared__ __align__(16) float sm[];
    float* bufP = sm + 2 * G::RH * RW;  // T ping-pongs between sm and sm + RH * RW

    const int S = A.steps;
    const int hy = S * HY, hx = S * HX;  // halo actually used by this launch
    const int SH = kHsTH + 2 * hy, SW = kHsTW + 2 * hx;
    int t = blockIdx.x;
    const int f = t / (A.tiles_x * A.tiles_y);
    t -= f * A.tiles_x * A.tiles_y;
    const int y0 = (t / A.tiles_x) * kHsTH, x0 = (t % A.tiles_x) * kHsTW;
    const int oy = y0 - hy, ox = x0 - hx;  // global coordinates of staged cell (0, 0)
    const float* T = A.t + (long long)f * A.fs;
    const float* Pw = A.p + (long long)f * A.fs;
    const int lo = -A.ntop, hi = A.h - 1 + A.nbot;  // valid rows (peer halo rows included)
    const bool border = oy < lo || ox < 0 || oy + SH > hi + 1 || ox + SW > A.w;

    // stage T and P over the tile + halo, clamped to the valid rows and the
    // image columns (rows of the staged box are spread over the threads,
    // columns over the lanes); rows beyond the stripe come from the peers
    for (int r = threadIdx.x / RW; r < SH; r += G::THREADS / RW) {
        const int c = threadIdx.x % RW;
        if (c < SW) {
            const int gy = min(max(oy + r, lo), hi), gx = min(max(ox + c, 0), A.w - 1);
            const float *srcT, *srcP;
            if (gy < 0) {
                const long long g = (long long)(A.ntop + gy) * A.ppitch + gx;
                srcT = A.ptop_t + g;
                srcP = A.ptop_p + g;
            } else if (gy >= A.h) {
                const long long g = (long long)(gy - A.h) * A.ppitch + gx;
                srcT = A.pbot_t + g;
                srcP = A.pbot_p + g;
            } else {
                const long long g = (long long)gy * A.pitch + gx;
                srcT = T + g;
                srcP = Pw + g;
            }
            sm[r * RW + c] = *srcT;
            bufP[r * RW + c] = *srcP;
        }
    }
    __syncthreads();

    const int col = threadIdx.x % RW, grp = threadIdx.x / RW;
    for (int k = 1; k <= S; ++k) {
        const float* cur = sm + ((k - 1) & 1) * (G::RH * RW);
        float* nxt = sm + (k & 1) * (G::RH * RW);
        // region of step k: the tile grown by (S - k) halo cells
        const int gyk = (S - k) * HY, gxk = (S - k) * HX;
        const int r0 = hy - gyk, c0 = hx - gxk;
        const int nr = kHsTH + 2 * gyk, nc = kHsTW + 2 * gxk;
        const bool last = k == S;
        const int c = c0 + col;
        if (col < nc) {
            const int half = (nr + 1) / 2;
            const int rs = r0 + grp * half, re = min(r0 + nr, rs + half);
            float win[3][2 * HX + 1];  // rows r-1, r, r+1 of columns c-HX..c+HX
            if (rs < re) {
#pragma unroll
                for (int a = -HY; a <= 0; ++a)
#pragma unroll
                    for (int b = -HX; b <= HX; ++b) win[a + 1][b + HX] = cur[(rs + a) * RW + c + b];
            }
#pragma unroll 4
            for (int r = rs; r < re; ++r) {
                if (HY) {
#pragma unroll
                    for (int b = -HX; b <= HX; ++b) win[2][b + HX] = cur[(r + 1) * RW + c + b];
                }
                // the 5-point HotSpot taps in the tile kernels' order (N, W, C, E, S);
                // the corners of the 3x3 are zero, and fmaf(0, x, acc) == acc
                float acc = 0.f;
#pragma unroll
                for (int a = -HY; a <= HY; ++a)
#pragma unroll
                    for (int b = -HX; b <= HX; ++b)
                        if (a == 0 || b == 0) acc = __fmaf_rn(A.w9[a + 1][b + 1], win[a + 1][b + HX], acc);
                acc = __fadd_rn(__fmaf_rn(A.alpha, bufP[r * RW + c], acc), A.beta);
                if (last) {
                    const int gy = oy + r, gx = ox + c;
                    if (gy < A.h && gx < A.w)
                        __stcs(A.out + (long long)f * A.fs + (long long)gy * A.pitch + gx, acc);
                } else {
                    nxt[r * RW + c] = acc;
                }
                if (HY) {
#pragma unroll
                    for (int b = 0; b < 2 * HX + 1; ++b) {
                        win[0][b] = win[1][b];
                        win[1][b] = win[2][b];
                    }
                } else if (r + 1 < re) {
#pragma unroll
                    for (int b = -HX; b <= HX; ++b) win[1][b + HX] = cur[(r + 1) * RW + c + b];
                }
            }
        }
        if (last) break;
        __syncthreads();
        // clamp-to-edge for the next step: out-of-image cells copy their edge cell
        if (border) {
            for (int idx = threadIdx.x; idx < nr * nc; idx += G::THREADS) {
                const int r = r0 + idx / nc, cc = c0 + idx % nc;
                const int gy = oy + r, gx = ox + cc;
                const int cy = min(max(gy, lo), hi), cx = min(max(gx, 0), A.w - 1);
                if (cy != gy || cx != gx) nxt[r * RW + cc] = nxt[(cy - oy) * RW + (cx - ox)];
            }
            __syncthreads();
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
    A.tiles_x = (v.w + kHsTW - 1) / kHsTW;
    A.tiles_y = (v.h + kHsTH - 1) / kHsTH;
    const long long nt = (long long)A.tiles_x * A.tiles_y * v.n;
    if (nt >= (1LL << 31)) return cudaErrorInvalidValue;
    auto launch = [&](auto kern, int smem, int threads) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        if (e != cudaSuccess) return e;
        kern<<<(unsigned)nt, threads, smem, s>>>(A);
        return cudaGetLastError();
    };
    cudaError_t e;
    if (p.hy && p.hx) e = launch(k_hotspot_tb<1, 1>, HsGeom<1, 1>::SMEM, HsGeom<1, 1>::THREADS);
    else if (p.hy) e = launch(k_hotspot_tb<1, 0>, HsGeom<1, 0>::SMEM, HsGeom<1, 0>::THREADS);
    else if (p.hx) e = launch(k_hotspot_tb<0, 1>, HsGeom<0, 1>::SMEM, HsGeom<0, 1>::THREADS);
    else e = launch(k_hotspot_tb<0, 0>, HsGeom<0, 0>::SMEM, HsGeom<0, 0>::THREADS);
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
