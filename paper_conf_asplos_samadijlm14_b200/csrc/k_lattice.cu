// k_lattice.cu -- the global-lattice reading of the stencil approximation
// (reading G): "Paraprox accesses a subset of
// values in the input array and replicates that subset to construct an
// approximate version of the array".  With a row reach
// d the accessed rows are the multiples of s = 2d+1; every row reads its
// nearest accessed row (rows past the last accessed one read the last), and
// the exact stencil is applied to that replicated array X~.
//
// This is the variant of the approximation that removes HBM bytes: only the
// accessed rows are ever read, 4/s + 4 bytes per output pixel instead of 8.
//
// Fast path (row lattice, square filters up to 9x9, dense or separable):
//  * A TMA tensor map over the accessed rows only ([n, A, w], row stride
//    s*pitch): each persistent CTA stages the AB accessed rows its output
//    tile needs (2-3-stage mbarrier ring, as in k_tiles.cuh).
//  * Output tiles are TH = 8 warps x RB rows with RB a multiple of s and tile
//    origins on multiples of s, so the phase y mod s of a thread's k-th output
//    row is k mod s -- a compile-time constant.  The filter rows that read the
//    same accessed row are folded on the host per phase (fp64 sums rounded to
//    fp32), so an output row costs (#accessed rows in its window) x K_x FMAs.
//  * Clamp-to-edge: the accessed-row index is clamped to [0, A-1] (this equals
//    clamping the window row first, then mapping it -- DESIGN.md); border
//    columns are replicated in shared memory.
// Column / centre lattices (no DRAM saving: a 32-byte sector holds 8 floats)
// and other shapes take k_lattice_generic: one thread per output, K_y x K_x
// gathered loads of X(g(clamp(y+i)), g(clamp(x+j))).
#include <climits>
#include <cstdlib>
#include <mutex>

#include "k_tiles.cuh"

constexpr int kLatMinBlocks = 2;  // CTAs per SM the register budget is sized for

namespace ppx {

constexpr int floor_div(int a, int b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }
// nearest accessed row of window row phi + i, relative: floor((phi+i)/s + 1/2)
constexpr int lat_m(int S, int t) { return floor_div(2 * t + S, 2 * S); }

// Warps per CTA: 4 for the dense lattices, 8 for the separable ones (r02
// kbench A/B of 4 against 8 warps: dense +1..+12 % except s = 3 / 7 at c4
// (-1..-2 %); separable -0.3..-1 %, profiles/r02_ab_w4.md)
template <bool SEP>
__host__ __device__ constexpr int lat_warps() { return SEP ? 8 : 4; }

template <int S, int R, int WARPS = kWarps>
struct LGeom {
    // rows per thread: a multiple of S near 8 (6 for S = 3: an even count for
    // the row-pair form below within the register budget of 2 CTAs per SM)
    static constexpr int RB = S == 3 ? 6 : S * ((8 + S / 2) / S > 0 ? (8 + S / 2) / S : 1);
    static constexpr int TH = WARPS * RB;                                      // tile rows
    static constexpr int QT = TH / S;                                          // row groups per tile
    static constexpr int QR = RB / S;                                          // row groups per thread
    static constexpr int MLO = lat_m(S, -R);
    static constexpr int MHI = lat_m(S, S - 1 + R);
    static constexpr int NA = MHI - MLO + 1;  // accessed-row slots per phase
    static constexpr int AB = QT + MHI - MLO; // staged accessed rows per tile
    static constexpr int HXP = round4(R);
    static constexpr int SW = kTW + 2 * HXP;
    static constexpr int STAGE_BYTES = SW * AB * 4;
    static constexpr int STAGE_STRIDE = (STAGE_BYTES + 127) & ~127;
    static constexpr int STAGES = (3 * STAGE_STRIDE <= 110 * 1024) ? 3 : 2;
    static constexpr int SMEM = STAGES * STAGE_STRIDE;
};

// does any filter row i in [-R, R] of phase phi read relative accessed row m?
template <int S, int R>
__host__ __device__ constexpr bool lat_used(int phi, int m) {
    for (int i = -R; i <= R; ++i)
        if (lat_m(S, phi + i) == m) return true;
    return false;
}

struct LatArgs {
    int n, h, w;
    int arows;  // accessed rows per frame (A)
    int tiles_x, tiles_y, ntiles;
    float* out;
    long long opitch, ofs;
    int stride, chunk;  // tile schedule, as TileArgs (bounded persistence)
    int step_f, step_ty, step_tx;  // the stride as (frames, tile rows, tile columns): TileWalk
    FastDiv dv_stride, dv_tpf, dv_tx;  // division by stride, tiles per frame, tiles_x (k_tiles.cuh)
};

// Row-pair form for the dense s = 3 lattice (the compute-bound one: 27-36
// FMAs per output for a 9x9 filter on 5.33 B/px): FFMA2 lanes hold output
// rows (y, y+1) of one column, as in k_tiles.cuh's row pairs; the staged
// value is the broadcast operand and the weight pair comes from wp, so no
// odd-column operand is rebuilt.  Per-output tap order (staged row, then
// column offset) is that of the column-pair form: bit-identical.
template <int S, bool SEP>
__host__ __device__ constexpr bool lat_row_pairs() { return !SEP && S == 3; }

struct LatW {
    // row pairs: wp[phi][m - MLO][b + 4] = (w[phi][m][b], w[phi'][m'][b]) with
    // (phi', m') the phase and relative accessed row of the next output row
    float2 wp[3][4][9];
    float w[9][4][9];  // dense: [phase][m - MLO][b + 4]
    float wy[9][4];    // separable: [phase][m - MLO]
    float wx[9];       // separable: [b + 4]
};

template <int S, int R, bool SEP>
__global__ void __launch_bounds__(32 * lat_warps<SEP>(), kLatMinBlocks * 8 / lat_warps<SEP>())
    k_lattice(const __grid_constant__ CUtensorMap tmap, const LatArgs A, const __grid_constant__ LatW W) {
    constexpr int WARPS = lat_warps<SEP>(), NT = 32 * WARPS;
    using G = LGeom<S, R, WARPS>;
    constexpr int HX = R, HXP = G::HXP, SW = G::SW, AB = G::AB, RB = G::RB, TH = G::TH, MLO = G::MLO;
    constexpr int NV = 4 + 2 * HXP;
    extern __shared__ __align__(128) unsigned char smem_raw[];
    __shared__ uint64_t bars[G::STAGES];

    const int tid = threadIdx.x, lane = tid & 31, wi = tid >> 5;
    const int tiles_per_frame = A.tiles_x * A.tiles_y;

    TileWalk wiss{}, wcur{};  // the issuing thread's walk (tiles ahead), every thread's walk (k_tiles.cuh)
    auto issue = [&](int s) {  // the tile at wiss
        fence_proxy_async();
        mbar_expect_tx(&bars[s], G::STAGE_BYTES);
        tma_load_3d(smem_raw + s * G::STAGE_STRIDE, &tmap, wiss.tx * kTW - HXP, wiss.ty * (TH / S) + MLO, wiss.f,
                    &bars[s]);
        wiss.step(A.step_f, A.step_ty, A.step_tx, A.tiles_x, A.tiles_y);
    };

    if (tid == 0) {
        for (int s = 0; s < G::STAGES; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
        tma_prefetch_desc(&tmap);
    }
    __syncthreads();
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    // CTA b takes tiles t_base + k * stride, k < chunk (k_tiles.cuh)
    const int wave = A.dv_stride.div((int)blockIdx.x);
    const long long t_base = (long long)wave * A.stride * A.chunk + ((int)blockIdx.x - wave * A.stride);
    const long long t_end = A.chunk == INT_MAX ? (long long)A.ntiles
                                               : min((long long)A.ntiles, (long long)(wave + 1) * A.stride * A.chunk);
    wcur.init((int)min(t_base, (long long)INT_MAX), A.dv_tpf, tiles_per_frame, A.dv_tx, A.tiles_x);
    wiss = wcur;
    if (tid == 0)
        for (int s = 0; s < G::STAGES - 1; ++s)
            if (t_base + (long long)s * A.stride < t_end) issue(s);

    int it = 0;
    for (long long tl = t_base; tl < t_end; tl += A.stride, ++it) {
        const int s = it % G::STAGES;
        if (tid == 0) {
            const long long ahead = tl + (long long)(G::STAGES - 1) * A.stride;
            if (ahead < t_end) issue((it + G::STAGES - 1) % G::STAGES);
        }
        const int f = wcur.f, y0 = wcur.ty * TH, x0 = wcur.tx * kTW;
        wcur.step(A.step_f, A.step_ty, A.step_tx, A.tiles_x, A.tiles_y);
        float* Sm = reinterpret_cast<float*>(smem_raw + s * G::STAGE_STRIDE);
        mbar_wait(&bars[s], (it / G::STAGES) & 1);

        const int a0 = y0 / S + MLO;  // accessed-row index of staged row 0
        const int rlo = max(0, -a0);
        const int rhi = min(AB - 1, A.arows - 1 - a0);
        const int clo = max(0, HXP - x0);
        const int chi = min(SW - 1, A.w - 1 - x0 + HXP);
        if (clo > 0 || chi < SW - 1) {  // border columns: replicate the edge (clamp)
            // only the out-of-image columns are touched: at most HXP per side
            const int nl = clo, nr = SW - 1 - chi, nb = nl + nr;
            for (int idx = tid; idx < AB * nb; idx += NT) {
                const int r = idx / nb, c = idx - r * nb;
                if (c < nl) Sm[r * SW + c] = Sm[r * SW + clo];
                else Sm[r * SW + chi + 1 + (c - nl)] = Sm[r * SW + chi];
            }
            __syncthreads();
        }

        const int tq0 = wi * G::QR;  // the thread's first row group (staged-row base)
        float2 acc[RB][2];
#pragma unroll
        for (int k = 0; k < RB; ++k) acc[k][0] = acc[k][1] = make_float2(0.f, 0.f);

        if constexpr (lat_row_pairs<S, SEP>()) {
            static_assert(RB % 2 == 0, "row pairs need an even RB");
            float2 rp[RB / 2][4];  // rp[p][c] = outputs (rows 2p, 2p+1) of column c
#pragma unroll
            for (int p = 0; p < RB / 2; ++p)
#pragma unroll
                for (int c = 0; c < 4; ++c) rp[p][c] = make_float2(0.f, 0.f);
            static_for<G::QR + G::NA - 1>([&](auto TT) {
                constexpr int tt = decltype(TT)::value;
                const int sr = min(max(tq0 + tt, rlo), rhi);
                float v[NV];
                const float4* p4 = reinterpret_cast<const float4*>(Sm + sr * SW) + lane;
#pragma unroll
                for (int q = 0; q < NV / 4; ++q) {
                    const float4 t = p4[q];
                    v[4 * q] = t.x, v[4 * q + 1] = t.y, v[4 * q + 2] = t.z, v[4 * q + 3] = t.w;
                }
                static_for<RB / 2>([&](auto KP) {
                    constexpr int p = decltype(KP)::value, k0 = 2 * p, k1 = 2 * p + 1;
                    constexpr int phi0 = k0 % S, m0 = tt - k0 / S + MLO;
                    constexpr int phi1 = k1 % S, m1 = tt - k1 / S + MLO;
                    constexpr bool u0 = m0 >= MLO && m0 <= G::MHI && lat_used<S, R>(phi0, m0);
                    constexpr bool u1 = m1 >= MLO && m1 <= G::MHI && lat_used<S, R>(phi1, m1);
                    if constexpr (u0 || u1) {
                        static_for<2 * HX + 1>([&](auto B) {
                            constexpr int b = decltype(B)::value - HX;
#pragma unroll
                            for (int c = 0; c < 4; ++c) {
                                const float xv = v[HXP + b + c];
                                if constexpr (u0 && u1)
                                    rp[p][c] = __ffma2_rn(W.wp[phi0][m0 - MLO][b + 4], make_float2(xv, xv), rp[p][c]);
                                else if constexpr (u0)
                                    rp[p][c].x = __fmaf_rn(W.w[phi0][m0 - MLO][b + 4], xv, rp[p][c].x);
                                else
                                    rp[p][c].y = __fmaf_rn(W.w[phi1][m1 - MLO][b + 4], xv, rp[p][c].y);
                            }
                        });
                    }
                });
            });
#pragma unroll
            for (int p = 0; p < RB / 2; ++p) {
                acc[2 * p][0] = make_float2(rp[p][0].x, rp[p][1].x);
                acc[2 * p][1] = make_float2(rp[p][2].x, rp[p][3].x);
                acc[2 * p + 1][0] = make_float2(rp[p][0].y, rp[p][1].y);
                acc[2 * p + 1][1] = make_float2(rp[p][2].y, rp[p][3].y);
            }
        } else if constexpr (!SEP) {
            static_for<G::QR + G::NA - 1>([&](auto TT) {
                constexpr int tt = decltype(TT)::value;  // staged row tq0 + tt
                const int sr = min(max(tq0 + tt, rlo), rhi);
                float2 ve[NV / 2], vo[NV / 2 - 1];
                load_pairs<NV>(Sm + sr * SW, lane, ve, vo);
                static_for<RB>([&](auto K) {
                    constexpr int k = decltype(K)::value;
                    constexpr int phi = k % S, m = tt - k / S + MLO;
                    if constexpr (m >= MLO && m <= G::MHI && lat_used<S, R>(phi, m)) {
                        static_for<2 * HX + 1>([&](auto B) {
                            constexpr int b = decltype(B)::value - HX;
                            fma_pairs<NV, HXP + b>(acc[k], W.w[phi][m - MLO][b + 4], ve, vo);
                        });
                    }
                });
            });
        } else {
            constexpr int RPT = (AB + WARPS - 1) / WARPS;
            float2 hz[RPT][2];
#pragma unroll
            for (int q = 0; q < RPT; ++q) {
                const int r = wi + q * WARPS;
                if (r < AB) {
                    const int sr = min(max(r, rlo), rhi);
                    float2 ve[NV / 2], vo[NV / 2 - 1];
                    load_pairs<NV>(Sm + sr * SW, lane, ve, vo);
                    hz[q][0] = hz[q][1] = make_float2(0.f, 0.f);
                    static_for<2 * HX + 1>([&](auto B) {
                        constexpr int b = decltype(B)::value - HX;
                        fma_pairs<NV, HXP + b>(hz[q], W.wx[b + 4], ve, vo);
                    });
                }
            }
            __syncthreads();
#pragma unroll
            for (int q = 0; q < RPT; ++q) {
                const int r = wi + q * WARPS;
                if (r < AB)
                    reinterpret_cast<float4*>(Sm + r * SW + HXP)[lane] =
                        make_float4(hz[q][0].x, hz[q][0].y, hz[q][1].x, hz[q][1].y);
            }
            __syncthreads();
            static_for<G::QR + G::NA - 1>([&](auto TT) {
                constexpr int tt = decltype(TT)::value;
                const float4 t = reinterpret_cast<const float4*>(Sm + (tq0 + tt) * SW + HXP)[lane];
                const float2 t0 = make_float2(t.x, t.y), t1 = make_float2(t.z, t.w);
                static_for<RB>([&](auto K) {
                    constexpr int k = decltype(K)::value;
                    constexpr int phi = k % S, m = tt - k / S + MLO;
                    if constexpr (m >= MLO && m <= G::MHI && lat_used<S, R>(phi, m)) {
                        const float wt = W.wy[phi][m - MLO];
                        const float2 w2 = make_float2(wt, wt);
                        acc[k][0] = __ffma2_rn(w2, t0, acc[k][0]);
                        acc[k][1] = __ffma2_rn(w2, t1, acc[k][1]);
                    }
                });
            });
        }

        const int x = x0 + 4 * lane;
        float* obase = A.out + (long long)f * A.ofs + x;
#pragma unroll
        for (int k = 0; k < RB; ++k) {
            const int y = y0 + wi * RB + k;
            if (y < A.h && x < A.w) {
                float* o = obase + (long long)y * A.opitch;
                if (x + 3 < A.w) {
                    __stcs(reinterpret_cast<float4*>(o), make_float4(acc[k][0].x, acc[k][0].y, acc[k][1].x, acc[k][1].y));
                } else {
                    const float r4[4] = {acc[k][0].x, acc[k][0].y, acc[k][1].x, acc[k][1].y};
#pragma unroll
                    for (int c = 0; c < 4; ++c)
                        if (x + c < A.w) __stcs(o + c, r4[c]);
                }
            }
        }
        __syncthreads();
    }
}

// ---- generic: any lattice, any filter, any layout ------------------------

struct LatTaps {
    int ky, kx;
    float w[kMaxTaps];
};

__device__ __forceinline__ int lat_g(int t, int d, int last) {
    if (d == 0) return t;
    const int s = 2 * d + 1;
    const int v = s * ((2 * t + s) / (2 * s));
    return v < last ? v : last;
}

__global__ void __launch_bounds__(256) k_lattice_generic(const float* __restrict__ in, View v, float* __restrict__ out,
                                                         long long opitch, long long ofs, int dy, int dx,
                                                         const __grid_constant__ LatTaps t) {
    const int x = blockIdx.x * blockDim.x + threadIdx.x;
    if (x >= v.w) return;
    const int lasty = dy ? (2 * dy + 1) * ((v.h - 1) / (2 * dy + 1)) : v.h - 1;
    const int lastx = dx ? (2 * dx + 1) * ((v.w - 1) / (2 * dx + 1)) : v.w - 1;
    const int ry = t.ky / 2, rx = t.kx / 2;
    // grid-stride over rows and frames: any h, n the ABI accepts launches
    for (int y = blockIdx.y * blockDim.y + threadIdx.y; y < v.h; y += gridDim.y * blockDim.y)
    for (int f = blockIdx.z; f < v.n; f += gridDim.z) {
        const float* F = in + (long long)f * v.fstride;
        float acc = 0.f;
        for (int i = -ry; i <= ry; ++i) {
            const int yy = lat_g(min(max(y + i, 0), v.h - 1), dy, lasty);
            for (int j = -rx; j <= rx; ++j) {
                const int xx = lat_g(min(max(x + j, 0), v.w - 1), dx, lastx);
                acc = fmaf(t.w[(i + ry) * t.kx + j + rx], __ldg(F + (long long)yy * v.pitch + xx), acc);
            }
        }
        out[(long long)f * ofs + (long long)y * opitch + x] = acc;
    }
}

// ---- registry / launch ---------------------------------------------------

using LatKernel = void (*)(const CUtensorMap, const LatArgs, const LatW);

struct LatInstance {
    int s, r;
    bool sep;
    LatKernel fn;
    int smem, ab, th, mlo, mhi;
    int threads;
    const char* name;
};

template <int S, int R, bool SEP>
LatInstance make_lat(const char* name) {
    using G = LGeom<S, R, lat_warps<SEP>()>;
    return LatInstance{S, R, SEP, k_lattice<S, R, SEP>, G::SMEM, G::AB, G::TH, G::MLO, G::MHI,
                       32 * lat_warps<SEP>(), name};
}

static const LatInstance* find_lat(int s, int r, bool sep) {
    static const LatInstance table[] = {
#define PPX_LAT(S, R)                                                  \
    make_lat<S, R, false>("lattice_dense_s" #S "_r" #R),               \
        make_lat<S, R, true>("lattice_sep_s" #S "_r" #R)
        PPX_LAT(3, 1), PPX_LAT(3, 2), PPX_LAT(3, 3), PPX_LAT(3, 4),
        PPX_LAT(5, 1), PPX_LAT(5, 2), PPX_LAT(5, 3), PPX_LAT(5, 4),
        PPX_LAT(7, 1), PPX_LAT(7, 2), PPX_LAT(7, 3), PPX_LAT(7, 4),
        PPX_LAT(9, 1), PPX_LAT(9, 2), PPX_LAT(9, 3), PPX_LAT(9, 4),
#undef PPX_LAT
    };
    for (const LatInstance& e : table)
        if (e.s == s && e.r == r && e.sep == sep) return &e;
    return nullptr;
}

// tiles per CTA (bounded persistence, k_tiles.cuh)
static int lattice_chunk() { return knobs().lattice_chunk; }

static bool lattice_force_generic() { return knobs().force_generic; }

static cudaError_t launch_lattice_generic(const paraprox_filter_s& lf, const float* in, const View& v, float* out,
                                          long long opitch, long long ofs, int dy, int dx, cudaStream_t s) {
    LatTaps t;
    t.ky = lf.ky;
    t.kx = lf.kx;
    for (int i = 0; i < lf.ky; ++i)
        for (int j = 0; j < lf.kx; ++j)
            t.w[i * lf.kx + j] = lf.separable ? lf.wy[i] * lf.wx[j] : lf.w[i * lf.kx + j];
    dim3 block(32, 8);
    const int gy = (v.h + 7) / 8;
    dim3 grid((v.w + 31) / 32, gy < 65535 ? gy : 65535, v.n < 65535 ? v.n : 65535);
    k_lattice_generic<<<grid, block, 0, s>>>(in, v, out, opitch, ofs, dy, dx, t);
    count_launch("lattice_generic");
    return cudaGetLastError();
}

cudaError_t launch_lattice(const paraprox_filter_s& lf, const float* in, const View& v, float* out, long long opitch,
                           long long ofs, int dy, int dx, cudaStream_t s) {
    const int r = lf.ky / 2;
    const LatInstance* e = nullptr;
    if (!lattice_force_generic() && dx == 0 && dy >= 1 && dy <= 4 && lf.ky == lf.kx && r >= 1 && r <= 4 &&
        v.lo == 0 && v.hi == v.h - 1 && !(reinterpret_cast<uintptr_t>(out) & 15) && !(opitch & 3) &&
        (v.n == 1 || !(ofs & 3)))
        e = find_lat(2 * dy + 1, r, lf.separable);
    if (!e) return launch_lattice_generic(lf, in, v, out, opitch, ofs, dy, dx, s);

    int dev = 0;
    cudaError_t err = cudaGetDevice(&dev);
    if (err != cudaSuccess) return err;
    const int S = e->s;
    const int arows = (v.h - 1) / S + 1;
    const long long fstride = v.n > 1 ? v.fstride : (long long)v.h * v.pitch;
    CUtensorMap tmap;
    // the accessed rows only: row stride s * pitch
    if (!encode_tmap_3d(&tmap, in, v.w, arows, v.n, (long long)S * v.pitch, fstride, kTW + 2 * round4(r), e->ab))
        return launch_lattice_generic(lf, in, v, out, opitch, ofs, dy, dx, s);
    static std::mutex mu;
    static int occ_cache[64][32] = {};
    static int sms[64] = {};
    const int idx = (int)(e - find_lat(3, 1, false));
    int occ = 0;
    {
        std::lock_guard<std::mutex> lk(mu);
        if (dev < 64 && idx >= 0 && idx < 32) occ = occ_cache[dev][idx];
        if (!occ) {
            err = cudaFuncSetAttribute(e->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, e->smem);
            if (err != cudaSuccess) return err;
            err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, e->fn, e->threads, e->smem);
            if (err != cudaSuccess) return err;
            if (occ < 1) occ = 1;
            if (dev < 64 && idx >= 0 && idx < 32) occ_cache[dev][idx] = occ;
        }
        if (dev < 64 && !sms[dev]) {
            err = cudaDeviceGetAttribute(&sms[dev], cudaDevAttrMultiProcessorCount, dev);
            if (err != cudaSuccess) return err;
        }
    }
    const int nsm = dev < 64 ? sms[dev] : 148;
    LatArgs A;
    A.n = v.n;
    A.h = v.h;
    A.w = v.w;
    A.arows = arows;
    A.tiles_x = (v.w + kTW - 1) / kTW;
    A.tiles_y = (v.h + e->th - 1) / e->th;
    const long long nt = (long long)A.tiles_x * A.tiles_y * v.n;
    if (nt >= (1LL << 31)) return launch_lattice_generic(lf, in, v, out, opitch, ofs, dy, dx, s);
    A.ntiles = (int)nt;
    A.out = out;
    A.opitch = opitch;
    A.ofs = ofs;
    // per-phase folded weights: filter rows i whose window row phi + i reads
    // accessed row m (relative) are summed (fp64, rounded once)
    LatW W = {};
    for (int phi = 0; phi < S; ++phi) {
        double acc[4][kMaxK] = {};
        double accy[4] = {};
        for (int i = -r; i <= r; ++i) {
            const int m = lat_m(S, phi + i) - e->mlo;
            if (lf.separable) {
                accy[m] += (double)lf.wy[i + r];
            } else {
                for (int j = 0; j < lf.kx; ++j) acc[m][j] += (double)lf.w[(i + r) * lf.kx + j];
            }
        }
        for (int m = 0; m <= e->mhi - e->mlo; ++m) {
            W.wy[phi][m] = (float)accy[m];
            for (int j = 0; j < lf.kx; ++j) W.w[phi][m][j - r + 4] = (float)acc[m][j];
        }
    }
    if (lf.separable)
        for (int j = 0; j < lf.kx; ++j) W.wx[j - r + 4] = lf.wx[j];
    if (S == 3 && !lf.separable)  // row-pair weights (lat_row_pairs)
        for (int phi = 0; phi < S; ++phi)
            for (int m = 0; m <= e->mhi - e->mlo; ++m) {
                const int phi1 = (phi + 1) % S, m1 = m - (phi == S - 1 ? 1 : 0);
                for (int b = 0; b < 9; ++b)
                    W.wp[phi][m][b] = make_float2(W.w[phi][m][b], m1 >= 0 ? W.w[phi1][m1][b] : 0.f);
            }
    const long long cap = (long long)nsm * occ;
    long long grid = nt < cap ? nt : cap;
    A.stride = (int)grid;
    A.chunk = lattice_chunk();
    {
        const long long tpf = (long long)A.tiles_x * A.tiles_y;
        A.step_f = (int)(A.stride / tpf);
        const long long r = A.stride - (long long)A.step_f * tpf;
        A.step_ty = (int)(r / A.tiles_x);
        A.step_tx = (int)(r - (long long)A.step_ty * A.tiles_x);
        A.dv_stride = make_fastdiv(A.stride);
        A.dv_tpf = make_fastdiv((int)tpf);
        A.dv_tx = make_fastdiv(A.tiles_x);
    }
    if (A.chunk != INT_MAX) {
        const long long waves = (nt + grid * A.chunk - 1) / (grid * A.chunk);
        if (waves * grid >= (1LL << 31)) return launch_lattice_generic(lf, in, v, out, opitch, ofs, dy, dx, s);
        grid *= waves;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(e->threads);
    cfg.dynamicSmemBytes = e->smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    err = cudaLaunchKernelEx(&cfg, e->fn, tmap, A, W);
    if (err != cudaSuccess) return err;
    count_launch(e->name);
    return cudaGetLastError();
}

}  // namespace ppx
