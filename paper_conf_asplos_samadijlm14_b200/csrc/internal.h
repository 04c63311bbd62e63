// internal.h -- shared declarations of libparaprox (host plan + kernel launchers).
// Not part of the ABI; see include/paraprox.h.
#pragma once

#include <cuda_runtime.h>

#include <atomic>
#include <cmath>
#include <cstdint>
#include <map>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "../../include/paraprox.h"

namespace ppx {

constexpr int kMaxK = PARAPROX_MAX_K;
constexpr int kMaxR = kMaxK / 2;            // 8
constexpr int kMaxTaps = kMaxK * kMaxK;     // 289

// One approximation plan: filter x per-axis reaching distances (dy, dx).
// Built once on the host and cached in the filter.
struct Plan {
    int ky = 1, kx = 1, ry = 0, rx = 0;
    bool separable = false;
    int dy = 0, dx = 0;                 // reaches, saturated to the radius
    int sy = 1, sx = 1;                 // reduction skipping rates (1 = none), saturated to K
    int my[kMaxK] = {}, mx[kMaxK] = {}; // index maps, m[i + r]
    int ny = 0, nx = 0;                 // |Ry|, |Rx| accessed offsets per axis
    int ay[kMaxK] = {}, ax[kMaxK] = {}; // accessed offsets, ascending
    int hy = 0, hx = 0;                 // halos = max |accessed offset|
    uint32_t masky = 0, maskx = 0;      // bit (a + kMaxR) set for accessed a
    int taps = 0;                       // ny*nx dense, ny+nx separable
    // folded weights: sum of the weights of every offset mapped to a rep,
    // accumulated in fp64 and rounded once to fp32
    float wf[kMaxTaps] = {};            // dense  [ny][nx]
    float wyf[kMaxK] = {}, wxf[kMaxK] = {}; // separable
};

struct Candidate {
    paraprox_scheme scheme;
    int reach;
    int dy, dx;
    int taps, hy, hx, sid;
};

}  // namespace ppx

struct paraprox_filter_s {
    int ky = 1, kx = 1;
    bool separable = false;
    std::vector<float> w;        // dense ky*kx
    std::vector<float> wy, wx;   // separable
    std::mutex mu;
    std::map<std::pair<int, int>, ppx::Plan> plans;
};

namespace ppx {

// ---- plan.cpp ----
int map_offset(int r, int d, int i);
const Plan& get_plan(paraprox_filter f, int dy, int dx);
// reduction approximation of the filter loops (§3.3.3): every sy-th
// filter row and sx-th filter column from the first, weights scaled by the rates
const Plan& get_plan_skip(paraprox_filter f, int sy, int sx);
bool is_skip_scheme(paraprox_scheme s);
void scheme_skips(paraprox_scheme s, int rate, int* sy, int* sx);
// candidates of the extended tuner: flags bit 0 stencil schemes, bit 1 reduction schemes
std::vector<Candidate> candidates_ex(paraprox_filter f, int flags);
void scheme_reaches(paraprox_scheme s, int reach, int* dy, int* dx);
std::vector<Candidate> candidates(paraprox_filter f);

// ---- device-side image view ----
struct View {
    int n, h, w;
    long long pitch, fstride;
    int lo, hi;  // valid input rows: [lo, hi] relative to row 0 (lo = -halo_top)
};

// An additive second input (HotSpot's power term, NEXT-4):
// out = stencil(in) + alpha * p[f, y, x] + beta, p laid out like the output.
struct Addend {
    const float* p = nullptr;
    long long pitch = 0, fstride = 0;
    float alpha = 0.f, beta = 0.f;
    int steps = 1;  // centre-only plans (k_pointwise): x <- w' x + alpha p + beta, `steps` times
};

// ---- kernels ----
// Each launcher enqueues on `s`, bumps the launch counter, records the kernel
// name and returns cudaGetLastError().
cudaError_t launch_stencil(const Plan& p, const float* in, const View& vin, float* out,
                           long long out_pitch, long long out_fstride, cudaStream_t s, const Addend* add = nullptr);
// global-lattice stencil (k_lattice.cu): exact stencil on the array rebuilt
// from the accessed rows/columns (reaches dy, dx); halos must be 0
cudaError_t launch_lattice(const paraprox_filter_s& f, const float* in, const View& v, float* out,
                           long long out_pitch, long long out_fstride, int dy, int dx, cudaStream_t s);
// temporally blocked HotSpot steps (k_hotspot.cu): `steps` <= kHotspotMaxSteps
// steps of a 3x3 plan plus the power term in one pass; t, p, out share v's
// layout (no halos)
constexpr int kHotspotMaxSteps = 8;
struct HotspotPeer {  // peer halo rows of a HotSpot row stripe (T and P), pitch in elements
    const float *top_t = nullptr, *top_p = nullptr, *bot_t = nullptr, *bot_p = nullptr;
    int ntop = 0, nbot = 0;
    long long pitch = 0;
};
cudaError_t launch_hotspot_tb(const Plan& p, const float* t, const float* pw, float* out, const View& v,
                              long long fs, float alpha, float beta, int steps, cudaStream_t s,
                              const HotspotPeer* peer = nullptr);
cudaError_t launch_flag_wait(const long long* flag, long long target, cudaStream_t s);
cudaError_t launch_flag_set(long long* flag, long long value, cudaStream_t s);
// Fused stencil + quality (the tuner's candidates, the runtime's checks): the
// plan's output is compared with `ref` (laid out like the output; ref_exact:
// ref holds the exact output, else the approximation) instead of being
// stored; 3 partials at d_part3 as launch_quality writes them.  *fused =
// false (nothing launched) when no fused kernel takes the plan and layout.
cudaError_t launch_stencil_quality(const Plan& p, const float* in, const View& vin, const float* ref,
                                   long long ref_pitch, long long ref_fstride, paraprox_metric m, bool ref_exact,
                                   double* d_part3, double* d_scratch, cudaStream_t s, bool* fused);
// Row-stripe stencil whose halo rows are read inside the kernel from peer
// pointers (CUDA IPC mappings of the neighbours' stripes): *taken = false
// when no tile instance takes the plan (the caller falls back to staging).
cudaError_t launch_stencil_peer(const Plan& p, const float* in, const View& v, float* out, long long opitch,
                                const float* htop, int ntop, const float* hbot, int nbot, long long hpitch,
                                cudaStream_t s, bool* taken);
bool fused_quality_enabled();  // PARAPROX_FUSED_QUALITY=0 turns the fused paths off
cudaError_t launch_quality_final(const double* d_scratch, int g, double count, paraprox_metric m, double* d_part3,
                                 cudaStream_t s);
cudaError_t launch_quality(const float* e, const float* a, const View& v, paraprox_metric m,
                           double* d_part3, double* d_scratch, cudaStream_t s);
constexpr int kQualityBlocks = 1184;  // partial-count cap of the persistent (tile, map) quality grids
// scratch (doubles) launch_quality and launch_stencil_quality need for an
// image of `count` pixels: one partial pair per CTA
// environment settings, read once (knobs.cpp)
struct Knobs {
    bool force_generic = false, fused_quality = true, tma_store = true, hotspot_tb = true;
    int tile_chunk = 0, lattice_chunk = 4;  // INT_MAX = fully persistent; tile 0 = per instance
};
const Knobs& knobs();
size_t quality_scratch_doubles(long long count);
// partial pairs that scratch holds (a quality grid must not exceed it)
size_t quality_scratch_pairs(long long count);

// ---- api.cpp helpers shared with runtime.cpp ----
#define PPX_CUDA(call)                                  \
    do {                                                \
        cudaError_t _e = (call);                        \
        if (_e != cudaSuccess) return cuda_fail(_e, #call); \
    } while (0)

paraprox_status fail(paraprox_status st, const std::string& msg);
paraprox_status cuda_fail(cudaError_t e, const char* where);
paraprox_status check_image(const paraprox_image* img, bool allow_halo);
View view_of(const paraprox_image* img);
bool overlaps(const float* in, const float* out, const paraprox_image* img);
paraprox_status run_stencil(paraprox_filter f, int dy, int dx, const float* in, float* out,
                            const paraprox_image* img, paraprox_stream s);
double quality_of(const double* p3, paraprox_metric m);
bool metric_ok(paraprox_metric m);
paraprox_status check_toq(double toq, paraprox_metric m);
cudaError_t scratch_alloc(void** p, size_t bytes, cudaStream_t s);
paraprox_status tune_partials_impl(paraprox_filter f, const float* d_train, const paraprox_image* img,
                                   paraprox_metric m, const std::vector<Candidate>& cands, double* h_partials,
                                   paraprox_stream s,
                                   double stop_toq = NAN);

// TMA-store epilogues of the tile and lattice kernels (default on);
// PARAPROX_TMA_STORE=0 keeps 128-bit register stores (A/B, and
// compute-sanitizer initcheck, which does not see bulk-tensor stores)
bool tma_store_enabled();

void count_launch(const char* name);
extern std::atomic<unsigned long long> g_launches;
extern thread_local const char* t_last_kernel;

}  // namespace ppx
