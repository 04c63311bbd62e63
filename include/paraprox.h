/*
 * paraprox.h -- C ABI of the B200-native Stencil & Partition approximation
 * library (libparaprox.so).
 *
 * The method: Samadi, Jamshidi, Lee, Mahlke, "Paraprox: Pattern-Based
 * Approximation for Data Parallel Applications", ASPLOS'14, §3.2 (PAPER.md
 * L1118-1226).  A K_y x K_x stencil (Gaussian, mean, convolution filter) is
 * approximated by reading only some elements of each output's tile: the
 * centre, one row, or one column stands in for its neighbours up to a
 * "reaching distance" (L1188-1218, Fig. 6), chosen by a runtime tuner so the
 * output quality (Table 1 metrics, L1644-1664) meets a target output quality
 * (TOQ, §4.2; runtime L572-592, training protocol L1620-1628).
 *
 * Conventions (all entry points):
 *  - Images are fp32, row-major.  A paraprox_image describes n frames of
 *    h x w elements; element (f, y, x) lives at base + f*frame_stride +
 *    y*pitch + x (elements, not bytes).  Input and output buffers share the
 *    descriptor.  Borders are clamped to the edge (reading S7).
 *  - halo_top / halo_bottom (input only): that many valid rows exist above
 *    row 0 / below row h-1 of every input frame (row-stripe decomposition);
 *    clamping happens at the edge of the valid rows, so an interior stripe
 *    with halos >= the filter radius computes exactly the rows the whole image
 *    would.  0 = clamp at that edge.  Outputs cover rows 0..h-1 only.
 *  - Device pointers ("d_") are caller-owned CUDA device memory; host
 *    pointers ("h_") are caller-owned host memory.  The library owns filter
 *    handles and nothing else; scratch comes from cudaMallocAsync on the
 *    caller's stream and is released before return (stream-ordered).
 *  - Streams: paraprox_stream is a cudaStream_t (NULL = legacy default
 *    stream).  Stencil calls are asynchronous with respect to the host;
 *    calls documented "syncs s" return after the stream has drained.
 *  - d_out must not overlap the input rows that are read (no in-place).
 *  - Errors are returned as paraprox_status codes; nothing aborts or throws.
 *    paraprox_last_error() gives a thread-local detail string.  Execution
 *    errors of asynchronous kernels surface at the caller's next sync.
 *  - There is no CPU fallback: every computation runs in this library's
 *    sm_100a kernels.
 */
#ifndef PARAPROX_H
#define PARAPROX_H

#ifdef __cplusplus
extern "C" {
#endif

#define PARAPROX_VERSION 1
#define PARAPROX_MAX_K 17 /* largest tile: the paper's 1x17 ConvSep loops (L1920-1922) */

#if defined(__GNUC__)
#define PARAPROX_API __attribute__((visibility("default")))
#else
#define PARAPROX_API
#endif

typedef struct CUstream_st* paraprox_stream;       /* == cudaStream_t */
typedef struct paraprox_filter_s* paraprox_filter; /* opaque, library-owned, immutable */
typedef struct paraprox_runtime_s* paraprox_runtime; /* opaque, library-owned runtime state */

typedef enum {
    PARAPROX_OK = 0,
    PARAPROX_ERR_INVALID_ARG = 1, /* null pointer, even/non-positive K, reach < 0,
                                     n/h/w < 1, pitch < w, overlap, bad TOQ, bad enum */
    PARAPROX_ERR_UNSUPPORTED = 2, /* K > PARAPROX_MAX_K */
    PARAPROX_ERR_CUDA = 3,        /* a CUDA runtime call or kernel launch failed */
    PARAPROX_ERR_ALLOC = 4        /* host or device allocation failed */
} paraprox_status;

/* Fig. 6 (L1156-1166): exact; row (rows within the reach copy the accessed
 * row); column; centre (the tile centre stands in for its neighbours).
 * The reduction approximation of the stencil's loops (§3.3.3,
 * applied to Convolution Separable's loops, L1920-1996; NEXT-3): skip-row
 * executes every N-th filter row (the vertical loop) and scales by N,
 * skip-col every N-th filter column, skip-both both loops; with these schemes
 * the "reach" argument is the skipping rate N >= 1 (1 = exact; rates above
 * the loop's trip count saturate to it). */
typedef enum {
    PARAPROX_EXACT = 0,
    PARAPROX_ROW = 1,
    PARAPROX_COL = 2,
    PARAPROX_CENTER = 3,
    PARAPROX_SKIP_ROW = 4,
    PARAPROX_SKIP_COL = 5,
    PARAPROX_SKIP_BOTH = 6
} paraprox_scheme;

/* Table 1 (L1644-1664): mean relative error (Gaussian, mean filters) and
 * L2-norm (Convolution Separable); quality = 1 - error.  PSNR (dB) is offered
 * as a reported metric and is not a paper metric (reading S11). */
typedef enum { PARAPROX_MRE = 0, PARAPROX_L2 = 1, PARAPROX_PSNR = 2 } paraprox_metric;

typedef struct {
    int n, h, w;             /* frames, rows, columns (>= 1)                 */
    long long pitch;         /* elements between rows (>= w)                 */
    long long frame_stride;  /* elements between frames
                                (>= (h + halo_top + halo_bottom) * pitch)     */
    int halo_top, halo_bottom; /* valid input rows above / below (>= 0)      */
} paraprox_image;

/* ---- filters ---------------------------------------------------------- */

/* Dense K_y x K_x weights, row-major, applied as a correlation (S8):
 * out(y,x) = sum_{i,j} w[i][j] * in(y + i - K_y/2, x + j - K_x/2).
 * K_y, K_x odd, 1..PARAPROX_MAX_K.  The weights are copied. */
PARAPROX_API paraprox_status paraprox_filter_create(int ky, int kx, const float* h_w, paraprox_filter* out);

/* Separable weights w = w_y (outer) w_x, computed as a fused horizontal then
 * vertical pass (ConvSep, Table 1).  The weights are copied. */
PARAPROX_API paraprox_status paraprox_filter_create_separable(int ky, const float* h_wy, int kx,
                                                 const float* h_wx, paraprox_filter* out);

PARAPROX_API void paraprox_filter_destroy(paraprox_filter f);

PARAPROX_API paraprox_status paraprox_filter_shape(paraprox_filter f, int* ky, int* kx, int* separable);

/* Plan introspection for per-axis reaches (reach_y, reach_x): the number of
 * taps the kernel evaluates (|Ry|*|Rx| dense, |Ry|+|Rx| separable), the
 * vertical/horizontal halo (largest accessed offset), and the per-axis index
 * maps m_y[0..K_y-1], m_x[0..K_x-1] (offset of the element read in place of
 * offset i - K/2; may be NULL).  Host-only. */
PARAPROX_API paraprox_status paraprox_plan_info(paraprox_filter f, int reach_y, int reach_x, int* taps,
                                   int* halo_y, int* halo_x, int* h_map_y, int* h_map_x);

/* ---- stencils (asynchronous on s) ------------------------------------- */

/* Exact stencil, every tap of every tile (the baseline, L544-552). */
PARAPROX_API paraprox_status paraprox_stencil_exact(paraprox_filter f, const float* d_in, float* d_out,
                                       const paraprox_image* img, paraprox_stream s);

/* Approximate stencil with a scheme and a reaching distance (L1188-1218).
 * reach > K/2 saturates; reach 0 or PARAPROX_EXACT computes the exact stencil.
 * Separable filters: row -> vertical pass approximated, column -> horizontal,
 * centre -> both ("reaching distances of both loops", L2110-2112). */
PARAPROX_API paraprox_status paraprox_stencil_approx(paraprox_filter f, paraprox_scheme scheme, int reach,
                                        const float* d_in, float* d_out,
                                        const paraprox_image* img, paraprox_stream s);

/* Per-axis reaching distances: row = (d, 0), column = (0, d), centre = (d, d). */
PARAPROX_API paraprox_status paraprox_stencil_approx_xy(paraprox_filter f, int reach_y, int reach_x,
                                           const float* d_in, float* d_out,
                                           const paraprox_image* img, paraprox_stream s);

/* Global-lattice reading (reading G):
 * "Paraprox accesses a subset of values in the input array and replicates
 * that subset to construct an approximate version of the array" (PAPER.md
 * L350-356).  Per axis with reach d >= 1 the accessed coordinates are the
 * multiples of s = 2d+1; every coordinate reads the nearest accessed one
 * (those past the last accessed one read the last), and the exact stencil is
 * applied to that array.  Schemes: row = (d, 0), column = (0, d), centre =
 * (d, d); reach 0 or EXACT = the exact stencil.  The row lattice reads only
 * every s-th row from HBM (4/s + 4 bytes per output pixel).  halo_top and
 * halo_bottom must be 0 (the lattice is anchored at row 0 of each frame).
 * Reaches above 2^20 are INVALID_ARG.  Asynchronous on s. */
PARAPROX_API paraprox_status paraprox_stencil_lattice(paraprox_filter f, paraprox_scheme scheme, int reach,
                                         const float* d_in, float* d_out,
                                         const paraprox_image* img, paraprox_stream s);
PARAPROX_API paraprox_status paraprox_stencil_lattice_xy(paraprox_filter f, int reach_y, int reach_x,
                                            const float* d_in, float* d_out,
                                            const paraprox_image* img, paraprox_stream s);

/* Reduction approximation with per-loop skipping rates (skip_y, skip_x >= 1;
 * rates above the loop's trip count saturate): every skip_y-th filter row
 * and skip_x-th filter column from the first, each loop scaled by its rate
 * (§3.3.3).  (1, 1) is the exact stencil. */
PARAPROX_API paraprox_status paraprox_stencil_skip_xy(paraprox_filter f, int skip_y, int skip_x,
                                         const float* d_in, float* d_out,
                                         const paraprox_image* img, paraprox_stream s);

/* Row stripe with peer halos (§8(e) P2; the B200-native form of the halo
 * exchange): the stencil of one stripe (img: n == 1, no halos) whose top_rows
 * rows directly above row 0 are read from d_top and bot_rows rows below row
 * h-1 from d_bot (pitch src_pitch elements) -- device pointers that may map a
 * neighbouring GPU's stripe over NVLink (paraprox_ipc_open), read inside the
 * stencil kernel with no separate collective.  0 rows = the image edge
 * (clamp).  Only the plan's halo h_y rows are read; a neighbour with
 * 0 < rows < h_y is INVALID_ARG (its first row is not the image edge, so no
 * clamp would be correct).  The caller orders the neighbours' writes before
 * this call (e.g. a barrier).  Asynchronous on s. */
PARAPROX_API paraprox_status paraprox_stencil_peer(paraprox_filter f, paraprox_scheme scheme, int reach,
                                      const float* d_in, float* d_out, const paraprox_image* img,
                                      const float* d_top, int top_rows, const float* d_bot, int bot_rows,
                                      long long src_pitch, paraprox_stream s);

/* CUDA IPC of device buffers between the processes of one node (one per GPU):
 * export writes a 64-byte handle of the allocation containing d_ptr and
 * d_ptr's byte offset in it; open maps a peer's handle (peer access enabled
 * lazily) and returns the allocation's base; close unmaps it. */
PARAPROX_API paraprox_status paraprox_ipc_export(const void* d_ptr, void* h_handle64, long long* offset);
PARAPROX_API paraprox_status paraprox_ipc_open(const void* h_handle64, void** d_base);
PARAPROX_API paraprox_status paraprox_ipc_close(void* d_base);

/* End-to-end convenience over HOST buffers: copies h_in to the device,
 * runs the stencil (scheme, reach), copies the result to h_out, overlapping
 * the transfers with the kernels chunk by chunk.  Pinned host memory gives
 * asynchronous copies; pageable memory works but serialises.  halo_top and
 * halo_bottom must be 0.  Syncs s. */
PARAPROX_API paraprox_status paraprox_run_host(paraprox_filter f, paraprox_scheme scheme, int reach,
                                  const float* h_in, float* h_out, const paraprox_image* img,
                                  paraprox_stream s);

/* ---- HotSpot: an iterated Stencil-Partition application (NEXT-4) -------- */

/* HotSpot (Table 1: 1024x1024, Stencil-Partition, MRE; 3x3 tiles,
 * L1916-1920).  `iterations` explicit thermal steps of the Rodinia kernel
 * (reading S25):
 *   T'(y,x) = T + c (P + (T_N + T_S - 2T) gy + (T_E + T_W - 2T) gx + (Tamb - T) gz)
 * with c = step_div_cap, gx = rx_inv, gy = ry_inv, gz = rz_inv; the 3x3 tile of
 * T read by each step is approximated by (scheme, reach) like a stencil (row:
 * the north/south reads take the centre row, ...).  d_temp, d_power and d_out
 * share img's layout (n independent grids); d_temp is not modified; halos are
 * allowed only with iterations == 1 (one step of a row stripe).  Scratch: one
 * image, stream-ordered.  Asynchronous on s. */
typedef struct {
    double step_div_cap, rx_inv, ry_inv, rz_inv, t_amb;
} paraprox_hotspot_params;
PARAPROX_API paraprox_status paraprox_hotspot(const paraprox_hotspot_params* prm, paraprox_scheme scheme,
                                 int reach, const float* d_temp, const float* d_power, float* d_out,
                                 const paraprox_image* img, int iterations, paraprox_stream s);

/* One HotSpot pass of `steps` (1..8) steps of a row stripe (img: n == 1, no
 * halos) whose neighbours' rows are read inside the blocked kernel from peer
 * pointers: the top_rows rows of temperature and power directly above row 0,
 * the bot_rows rows below row h-1 (pitch src_pitch; 0 rows = the image edge).
 * A pass needs steps x h_y rows from each peer (h_y = 1 for the exact and
 * column schemes, 0 for row and centre).  The caller orders the passes across
 * GPUs (paraprox_flag_wait / _set).  Asynchronous on s. */
PARAPROX_API paraprox_status paraprox_hotspot_peer(const paraprox_hotspot_params* prm, paraprox_scheme scheme,
                                      int reach, const float* d_temp, const float* d_power, float* d_out,
                                      const paraprox_image* img, int steps, const float* d_top_temp,
                                      const float* d_top_power, int top_rows, const float* d_bot_temp,
                                      const float* d_bot_power, int bot_rows, long long src_pitch,
                                      paraprox_stream s);

/* Device-side ordering across GPUs (the flag may be a peer GPU's memory
 * mapped by paraprox_ipc_open): wait enqueues a kernel that spins (acquire,
 * system scope) until *d_flag >= target; set enqueues a release store of
 * value after the preceding work of s.  Asynchronous on s. */
PARAPROX_API paraprox_status paraprox_flag_wait(const long long* d_flag, long long target, paraprox_stream s);
PARAPROX_API paraprox_status paraprox_flag_set(long long* d_flag, long long value, paraprox_stream s);

/* ---- output quality (syncs s) ------------------------------------------ */

/* Quality of d_approx against d_exact over all n*h*w elements (pooled over
 * frames, S12): 1 - MRE, 1 - L2 or PSNR dB.  fp64 accumulation in a fixed
 * order: the result is deterministic for a given image shape. */
PARAPROX_API paraprox_status paraprox_quality(const float* d_exact, const float* d_approx,
                                 const paraprox_image* img, paraprox_metric m,
                                 double* h_quality, paraprox_stream s);

/* The 3 fp64 partial sums behind paraprox_quality (MRE: sum of relative
 * errors, count, 0; L2: sum (A-E)^2, sum E^2, count; PSNR: sum (A-E)^2,
 * count, 0).  Partials of disjoint pixel sets add (multi-GPU all-reduce). */
PARAPROX_API paraprox_status paraprox_quality_partials(const float* d_exact, const float* d_approx,
                                          const paraprox_image* img, paraprox_metric m,
                                          double* h_partials3, paraprox_stream s);

/* Asynchronous variant: the 3 partials are written to caller-owned device
 * memory d_partials3 (3 doubles) in stream order; nothing is copied to the
 * host and the stream is not synchronised (runtime quality checks inside a
 * pipeline or a CUDA graph).  Same partials, bit for bit, as
 * paraprox_quality_partials. */
PARAPROX_API paraprox_status paraprox_quality_partials_async(const float* d_exact, const float* d_approx,
                                                const paraprox_image* img, paraprox_metric m,
                                                double* d_partials3, paraprox_stream s);

/* Quality from (summed) partials.  Host-only. */
PARAPROX_API paraprox_status paraprox_quality_from_partials(const double* h_partials3, paraprox_metric m,
                                               double* h_quality);

/* ---- TOQ tuner (syncs s) ------------------------------------------------ */

/* The runtime tuner (L572-592; L1220-1226; training on the first frames,
 * L1620-1628): the exact kernel runs once on the training frames d_train,
 * then the candidates (scheme, reach) run in cost order, each scored against
 * it; the first candidate with quality >= toq is returned (the scan stops
 * there: one stream sync per candidate scored), else (EXACT, 0, 1.0 or
 * +inf dB).  toq in (0, 1] for MRE / L2; any value (dB) for PSNR.  The
 * decision equals paraprox_tune_decide on paraprox_tune_partials' full scan. */
PARAPROX_API paraprox_status paraprox_tune(paraprox_filter f, const float* d_train, const paraprox_image* img,
                              double toq, paraprox_metric m, paraprox_scheme* out_scheme,
                              int* out_reach, double* out_quality, paraprox_stream s);

/* Candidates in cost order (O7).  *n receives the count; at most
 * cap entries are written (schemes/reaches may be NULL to query the count). */
PARAPROX_API paraprox_status paraprox_tune_candidates(paraprox_filter f, int cap, int* n,
                                         paraprox_scheme* schemes, int* reaches);

/* Multi-GPU split of paraprox_tune: 3 quality partials per candidate (in
 * candidate order, 3*n doubles) for the local training frames ... */
PARAPROX_API paraprox_status paraprox_tune_partials(paraprox_filter f, const float* d_train,
                                       const paraprox_image* img, paraprox_metric m,
                                       double* h_partials, paraprox_stream s);

/* ... and the host-only decision from (all-reduced) partials.  Every rank
 * holding the same summed partials reaches the same decision. */
PARAPROX_API paraprox_status paraprox_tune_decide(paraprox_filter f, const double* h_partials,
                                     paraprox_metric m, double toq, paraprox_scheme* out_scheme,
                                     int* out_reach, double* out_quality);

/* Extended tuner over the stencil schemes (flags bit 0) and the reduction
 * schemes (flags bit 1: skip-both / skip-row / skip-col with rates 2..r+1),
 * one integer cost order over both (O7 + S24).  flags = 1 is
 * paraprox_tune.  Same conventions as the functions above; the returned
 * "reach" is the skipping rate for the reduction schemes. */
PARAPROX_API paraprox_status paraprox_tune_ex(paraprox_filter f, int flags, const float* d_train,
                                 const paraprox_image* img, double toq, paraprox_metric m,
                                 paraprox_scheme* out_scheme, int* out_reach, double* out_quality,
                                 paraprox_stream s);
PARAPROX_API paraprox_status paraprox_tune_candidates_ex(paraprox_filter f, int flags, int cap, int* n,
                                            paraprox_scheme* schemes, int* reaches);
PARAPROX_API paraprox_status paraprox_tune_partials_ex(paraprox_filter f, int flags, const float* d_train,
                                          const paraprox_image* img, paraprox_metric m,
                                          double* h_partials, paraprox_stream s);
PARAPROX_API paraprox_status paraprox_tune_decide_ex(paraprox_filter f, int flags, const double* h_partials,
                                        paraprox_metric m, double toq, paraprox_scheme* out_scheme,
                                        int* out_reach, double* out_quality);

/* Lattice tuner: the exact stencil once on d_train, then the row lattice
 * with reach 4, 3, 2, 1 (fewest HBM bytes first); the first whose quality
 * >= toq wins, else (EXACT, 0, 1.0 / +inf dB).  Syncs s.  Its multi-GPU split:
 * 3 partials per candidate (12 doubles, candidate order) for the local
 * frames, then a host-only decision from the (all-reduced) partials. */
PARAPROX_API paraprox_status paraprox_tune_lattice(paraprox_filter f, const float* d_train,
                                      const paraprox_image* img, double toq, paraprox_metric m,
                                      paraprox_scheme* out_scheme, int* out_reach, double* out_quality,
                                      paraprox_stream s);
PARAPROX_API paraprox_status paraprox_tune_lattice_partials(paraprox_filter f, const float* d_train,
                                               const paraprox_image* img, paraprox_metric m,
                                               double* h_partials12, paraprox_stream s);
PARAPROX_API paraprox_status paraprox_tune_lattice_decide(const double* h_partials12, paraprox_metric m,
                                             double toq, paraprox_scheme* out_scheme, int* out_reach,
                                             double* out_quality);

/* ---- runtime: periodic quality check and back-off (NEXT-2) ------------ */

/* The runtime loop of PAPER.md L572-592 ("checks the output quality
 * periodically ... If the quality drops below the TOQ, it uses a less
 * aggressive approximation"; every 40-50 invocations keeps the overhead under
 * 5 %, L2656-2666).  DESIGN.md readings R1-R4:
 *  - train: the TOQ tuner on d_train picks rung 0; the ladder continues with
 *    the later candidates (cost order) whose training quality is higher than
 *    every earlier rung, and ends at EXACT;
 *  - run: the current rung's stencil into d_out (asynchronous on s); on the
 *    1st and then every check_every-th invocation (0 = never) the exact
 *    stencil of the same input and the quality of d_out against it are also
 *    enqueued on s, their partials copied to pinned host memory behind an
 *    event -- the call does not wait for them;
 *  - a finished check (seen at the next run, or forced by _sync) with quality
 *    < toq moves one rung down the ladder.
 * The runtime owns its check buffers (device memory of one output image,
 * allocated at the first check); the filter must outlive it.  Not for
 * concurrent use from several threads on different streams (calls are
 * serialised by a mutex). */
PARAPROX_API paraprox_status paraprox_runtime_create(paraprox_filter f, double toq, paraprox_metric m,
                                        int check_every, paraprox_runtime* out);
PARAPROX_API void paraprox_runtime_destroy(paraprox_runtime rt);
/* Syncs s. */
PARAPROX_API paraprox_status paraprox_runtime_train(paraprox_runtime rt, const float* d_train,
                                       const paraprox_image* img, paraprox_stream s);
PARAPROX_API paraprox_status paraprox_runtime_run(paraprox_runtime rt, const float* d_in, float* d_out,
                                     const paraprox_image* img, paraprox_stream s);
/* Waits for a pending check and applies it. */
PARAPROX_API paraprox_status paraprox_runtime_sync(paraprox_runtime rt);
/* Current rung and counters (host-only; any pointer may be NULL). */
PARAPROX_API paraprox_status paraprox_runtime_state(paraprox_runtime rt, paraprox_scheme* scheme, int* reach,
                                       long long* invocations, long long* checks, long long* backoffs,
                                       double* last_quality);
/* Profiled training (call before _train; the paper's runtime "profiles the
 * kernels and picks ... the best performance"): every candidate
 * that meets the TOQ on the training frames, and the exact stencil, is timed
 * there (CUDA events, best of 3); rung 0 is the fastest passing candidate and
 * the ladder continues with the passing candidates of strictly higher
 * training quality, then EXACT.  Not bit-reproducible across runs (timings). */
PARAPROX_API paraprox_status paraprox_runtime_set_profiled(paraprox_runtime rt, int enable);
/* Measured ms per candidate in tuner order, then the exact stencil (NaN where
 * not measured); *n = candidates + 1. */
PARAPROX_API paraprox_status paraprox_runtime_timings(paraprox_runtime rt, int cap, int* n, double* ms);
/* The ladder: *n rungs, at most cap written (arrays may be NULL). */
PARAPROX_API paraprox_status paraprox_runtime_ladder(paraprox_runtime rt, int cap, int* n,
                                        paraprox_scheme* schemes, int* reaches, double* train_quality);

/* ---- diagnostics -------------------------------------------------------- */

PARAPROX_API const char* paraprox_status_string(paraprox_status st);
PARAPROX_API const char* paraprox_last_error(void);       /* thread-local detail of the last failure */
PARAPROX_API int paraprox_version(void);
/* Kernels this library has launched since load (all threads). */
PARAPROX_API unsigned long long paraprox_launch_count(void);
/* Name of the kernel variant the last stencil call on this thread used. */
PARAPROX_API const char* paraprox_last_kernel(void);

#ifdef __cplusplus
}
#endif
#endif /* PARAPROX_H */
