// dispatch.cu -- picks the kernel variant for a plan and an image layout.
//
// Centre-only plans (full collapse, or 1x1 filters) are maps: k_pointwise.cu.
// Fast path: the persistent TMA tile kernel instance (k_tiles.cuh) whose
// compile-time accessed-offset masks equal the plan's (every plan of a filter
// up to 9x9 has one; instances are registered by inst_r*_*.cu).  It needs a
// layout TMA can describe (16-byte aligned rows) and 16-byte aligned output
// rows.  Anything else takes the generic kernel (k_generic.cu): slower, same
// results, still on the GPU.
#include <climits>
#include <cstdlib>
#include <mutex>
#include <vector>

#include "k_tiles.cuh"

namespace ppx {

cudaError_t launch_generic(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                           long long ofs, cudaStream_t s, const Addend* add);
cudaError_t launch_pointwise(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                             long long ofs, cudaStream_t s, const Addend* add);
bool launch_pointwise_quality(const Plan& p, const float* in, const View& v, const float* ref, long long rpitch,
                              long long rfs, int metric, int ref_exact, double* part, int* grid_out, cudaStream_t s,
                              cudaError_t* err);

struct PeerHalo {
    const float* top;
    const float* bot;
    int ntop, nbot;
    long long pitch;
};

struct QualityOut {
    const float* ref;
    long long rpitch, rfs;
    int metric, ref_exact;
    double* part;
    long long cap_pairs;  // partial pairs the scratch holds (quality_scratch_pairs)
    int grid;             // written: CTAs that wrote partials
};

void register_r1_dense();
void register_r2_dense();
void register_r3_dense();
void register_r4_dense();
void register_r1_sep();
void register_r2_sep();
void register_r3_sep();
void register_r4_sep();
void register_r8_sep();

namespace {

constexpr int kMaxDev = 64;

struct Entry {
    TileInstance ti;
    bool ready[kMaxDev] = {};
    int occ[kMaxDev] = {};   // plain instance
    int occq[kMaxDev] = {};  // fused-quality instance
};

std::vector<Entry>& reg() {
    static std::vector<Entry> r;
    return r;
}

std::mutex g_mu;
int g_sms[kMaxDev] = {};

void init_registry() {
    static std::once_flag once;
    std::call_once(once, [] {
        register_r1_dense();
        register_r2_dense();
        register_r3_dense();
        register_r4_dense();
        register_r1_sep();
        register_r2_sep();
        register_r3_sep();
        register_r4_sep();
        register_r8_sep();
    });
}

bool force_generic() { return knobs().force_generic; }

}  // namespace

// tiles per CTA of the plain tile kernels (k_tiles.cuh, bounded persistence)
// (r02 kbench sweep of 1, 2, 3, 4, 6, 16: 4-warp instances +3..+11 % at 4
// against 16 on c1-c4; 8-warp instances -2..-9 % below 16)
static int tile_chunk(int threads) {
    const int k = knobs().tile_chunk;
    return k ? k : (threads <= 128 ? 4 : 16);
}

bool tma_store_enabled() { return knobs().tma_store; }

void register_tile_instance(const TileInstance& ti) {
    for (const Entry& o : reg())  // the same instance serves several radii
        if (o.ti.fn == ti.fn) return;
    Entry e;
    e.ti = ti;
    reg().push_back(e);
}

static cudaError_t launch_tiles(Entry& e, const Plan& p, const float* in, const View& v, float* out,
                                long long opitch, long long ofs, cudaStream_t s, const Addend* add, bool* taken,
                                QualityOut* qo = nullptr, const PeerHalo* ph = nullptr) {
    *taken = false;
    int dev = 0;
    cudaError_t err = cudaGetDevice(&dev);
    if (err != cudaSuccess) return err;
    if (dev >= kMaxDev) return cudaSuccess;
    // layout checks: TMA-describable input, 16-byte aligned output rows
    if ((reinterpret_cast<uintptr_t>(out) & 15) || (opitch & 3) || (v.n > 1 && (ofs & 3))) return cudaSuccess;
    if (add && ((reinterpret_cast<uintptr_t>(add->p) & 15) || (add->pitch & 3) || (v.n > 1 && (add->fstride & 3))))
        return cudaSuccess;
    const int rows_valid = v.hi - v.lo + 1;
    const long long fstride = v.n > 1 ? v.fstride : (long long)rows_valid * v.pitch;
    CUtensorMap tmap;
    const int box_w = e.ti.sw, box_h = e.ti.th + 2 * e.ti.hy;
    if (!encode_tmap_3d(&tmap, in + (long long)v.lo * v.pitch, v.w, rows_valid, v.n, v.pitch, fstride, box_w, box_h))
        return cudaSuccess;
    // output map for the TMA-store epilogue (PARAPROX_TMA_STORE); a layout it
    // cannot describe keeps the register-store epilogue
    CUtensorMap omap = tmap;  // (unused unless A.tma_store)
    const bool tma_store = !qo && !add && tma_store_enabled() &&
                           encode_tmap_3d(&omap, out, v.w, v.h, v.n, opitch, v.n > 1 ? ofs : (long long)v.h * opitch,
                                          kTW, e.ti.store_rows);
    {
        std::lock_guard<std::mutex> lk(g_mu);
        if (!e.ready[dev]) {
            int occ = 0, occq = 0;
            for (TileKernel fn : {e.ti.fn, e.ti.fnq}) {
                err = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, e.ti.smem);
                if (err != cudaSuccess) return err;
                err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(fn == e.ti.fn ? &occ : &occq, fn, e.ti.threads,
                                                                    e.ti.smem);
                if (err != cudaSuccess) return err;
            }
            if (!g_sms[dev]) {
                err = cudaDeviceGetAttribute(&g_sms[dev], cudaDevAttrMultiProcessorCount, dev);
                if (err != cudaSuccess) return err;
            }
            e.occ[dev] = occ > 0 ? occ : 1;
            e.occq[dev] = occq > 0 ? occq : 1;
            e.ready[dev] = true;
        }
    }
    TileArgs A;
    A.n = v.n;
    A.h = v.h;
    A.w = v.w;
    A.rows_valid = rows_valid;
    A.row_off = -v.lo;
    A.tiles_x = (v.w + kTW - 1) / kTW;
    A.tiles_y = (v.h + e.ti.th - 1) / e.ti.th;
    const long long nt = (long long)A.tiles_x * A.tiles_y * v.n;
    if (nt >= (1LL << 31)) return cudaSuccess;
    A.ntiles = (int)nt;
    A.out = out;
    A.opitch = opitch;
    A.ofs = ofs;
    A.addp = add ? add->p : nullptr;
    A.apitch = add ? add->pitch : 0;
    A.afs = add ? add->fstride : 0;
    A.alpha = add ? add->alpha : 0.f;
    A.beta = add ? add->beta : 0.f;
    A.refp = qo ? qo->ref : nullptr;
    A.rpitch = qo ? qo->rpitch : 0;
    A.rfs = qo ? qo->rfs : 0;
    A.metric = qo ? qo->metric : 0;
    A.ref_exact = qo ? qo->ref_exact : 0;
    A.part = qo ? qo->part : nullptr;
    A.htop = ph ? ph->top : nullptr;
    A.hbot = ph ? ph->bot : nullptr;
    A.ntop = ph ? ph->ntop : 0;
    A.nbot = ph ? ph->nbot : 0;
    A.hpitch = ph ? ph->pitch : 0;
    A.tma_store = tma_store ? 1 : 0;
    if (qo && ((reinterpret_cast<uintptr_t>(qo->ref) & 15) || (qo->rpitch & 3) || (v.n > 1 && (qo->rfs & 3))))
        return cudaSuccess;
    TapW W = {};
    if (p.separable) {
        for (int i = 0; i < p.ny; ++i) W.wy[p.ay[i] + 8] = p.wyf[i];
        for (int j = 0; j < p.nx; ++j) W.wx[p.ax[j] + 8] = p.wxf[j];
        for (int b = 1; b < 17; ++b) {  // weight pairs of the wide separable path
            W.wxp[b] = make_float2(W.wx[b], W.wx[b - 1]);
            W.wyp[b] = make_float2(W.wy[b], W.wy[b - 1]);
        }
    } else {
        for (int i = 0; i < p.ny; ++i)
            for (int j = 0; j < p.nx; ++j) W.w[p.ay[i] + 4][p.ax[j] + 4] = p.wf[i * p.nx + j];
        for (int a = -3; a <= 4; ++a)  // row-pair weights (k_tiles.cuh, use_row_pairs)
            for (int b = 0; b < 9; ++b) W.wp[a + 4][b] = make_float2(W.w[a + 4][b], W.w[a + 3][b]);
    }
    long long cap = (long long)g_sms[dev] * (qo ? e.occq[dev] : e.occ[dev]);
    if (qo && cap > kQualityBlocks) cap = kQualityBlocks;  // one partial pair per CTA
    int grid = (int)(nt < cap ? nt : cap);
    // bounded persistence (k_tiles.cuh) for the HBM-bound instances: on 8.5 GB
    // (c3) chunks of 16 tiles cut the exact 7x7's DRAM reads from 1.32x to
    // 1.02x the input and run 29 % faster; FMA-bound plans (> 45 FMAs per
    // pixel at 1965 MHz) lose ~3 % to CTA restarts and stay
    // persistent.  A wave of `grid` CTAs takes grid * chunk tiles.
    const int taps = p.separable ? p.ny + p.nx : p.ny * p.nx;
    A.stride = grid;
    A.chunk = taps > 45 ? INT_MAX : tile_chunk(e.ti.threads);
    if (A.chunk != INT_MAX) {
        const long long waves = (nt + (long long)grid * A.chunk - 1) / ((long long)grid * A.chunk);
        if (waves * grid >= (1LL << 31)) return cudaSuccess;
        if (qo && waves * grid > qo->cap_pairs) {
            // one partial pair per CTA: when the tiles outnumber the pixels'
            // share of the scratch (many tiny frames, w < 8), keep the
            // persistent grid (<= kQualityBlocks pairs, always in the scratch)
            A.chunk = INT_MAX;
        } else {
            grid = (int)(waves * grid);
        }
    }
    if (qo) qo->grid = grid;  // one partial pair per CTA, grid <= qo->cap_pairs
    {  // the stride as (frames, tile rows, tile columns): the kernel's TileWalk
        const long long tpf = (long long)A.tiles_x * A.tiles_y;
        A.step_f = (int)(A.stride / tpf);
        const long long r = A.stride - (long long)A.step_f * tpf;
        A.step_ty = (int)(r / A.tiles_x);
        A.step_tx = (int)(r - (long long)A.step_ty * A.tiles_x);
        A.dv_stride = make_fastdiv(A.stride);
        A.dv_tpf = make_fastdiv((int)tpf);
        A.dv_tx = make_fastdiv(A.tiles_x);
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(e.ti.threads);
    cfg.dynamicSmemBytes = e.ti.smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    err = cudaLaunchKernelEx(&cfg, qo ? e.ti.fnq : e.ti.fn, tmap, A, W, omap);
    if (err != cudaSuccess) return err;
    count_launch(qo ? "tile_quality" : e.ti.name);
    *taken = true;
    return cudaGetLastError();
}

cudaError_t launch_stencil(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                           long long ofs, cudaStream_t s, const Addend* add) {
    // a plan that accesses only the centre is a map: stream it (k_pointwise.cu)
    if (!force_generic() && p.hy == 0 && p.hx == 0) return launch_pointwise(p, in, v, out, opitch, ofs, s, add);
    const int rmax = p.separable ? 8 : 4;  // tile instances: dense r <= 4, separable r <= 8
    if (!force_generic() && p.ry <= rmax && p.rx <= rmax) {
        init_registry();
        for (Entry& e : reg()) {
            if (e.ti.sep != p.separable || e.ti.masky != p.masky || e.ti.maskx != p.maskx) continue;
            bool taken = false;
            cudaError_t err = launch_tiles(e, p, in, v, out, opitch, ofs, s, add, &taken);
            if (err != cudaSuccess || taken) return err;
            break;
        }
    }
    return launch_generic(p, in, v, out, opitch, ofs, s, add);
}

cudaError_t launch_stencil_quality(const Plan& p, const float* in, const View& v, const float* ref,
                                   long long ref_pitch, long long ref_fstride, paraprox_metric m, bool ref_exact,
                                   double* d_part3, double* d_scratch, cudaStream_t s, bool* fused) {
    *fused = false;
    if (force_generic()) return cudaSuccess;
    const double count = (double)v.n * (double)v.h * (double)v.w;
    if (p.hy == 0 && p.hx == 0) {
        int grid = 0;
        cudaError_t err = cudaSuccess;
        if (!launch_pointwise_quality(p, in, v, ref, ref_pitch, ref_fstride, (int)m, ref_exact ? 1 : 0, d_scratch,
                                      &grid, s, &err))
            return cudaSuccess;
        if (err != cudaSuccess) return err;
        *fused = true;
        return launch_quality_final(d_scratch, grid, count, m, d_part3, s);
    }
    const int rmax = p.separable ? 8 : 4;
    if (p.ry > rmax || p.rx > rmax) return cudaSuccess;
    init_registry();
    for (Entry& e : reg()) {
        if (e.ti.sep != p.separable || e.ti.masky != p.masky || e.ti.maskx != p.maskx) continue;
        QualityOut qo{ref, ref_pitch, ref_fstride, (int)m, ref_exact ? 1 : 0, d_scratch,
                      (long long)quality_scratch_pairs((long long)v.n * v.h * v.w), 0};
        bool taken = false;
        // the output pointer only fixes the layout checks: nothing is stored
        cudaError_t err = launch_tiles(e, p, in, v, const_cast<float*>(ref), ref_pitch, ref_fstride, s, nullptr,
                                       &taken, &qo);
        if (err != cudaSuccess) return err;
        if (!taken) return cudaSuccess;
        *fused = true;
        return launch_quality_final(d_scratch, qo.grid, count, m, d_part3, s);
    }
    return cudaSuccess;
}

cudaError_t launch_stencil_peer(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                                const float* htop, int ntop, const float* hbot, int nbot, long long hpitch,
                                cudaStream_t s, bool* taken) {
    *taken = false;
    if (force_generic() || v.n != 1 || v.lo != 0 || v.hi != v.h - 1) return cudaSuccess;
    const int rmax = p.separable ? 8 : 4;
    if (p.ry > rmax || p.rx > rmax) return cudaSuccess;
    init_registry();
    const PeerHalo ph{htop, hbot, ntop, nbot, hpitch};
    for (Entry& e : reg()) {
        if (e.ti.sep != p.separable || e.ti.masky != p.masky || e.ti.maskx != p.maskx) continue;
        return launch_tiles(e, p, in, v, out, opitch, (long long)v.h * opitch, s, nullptr, taken, nullptr, &ph);
    }
    return cudaSuccess;
}

}  // namespace ppx
