// plan.cpp -- host side of the approximation: the
// reaching-distance index maps, the accessed (representative) offsets, the
// halos, the folded tap weights and the tuner's candidate order.
//
// PAPER.md §3.2.3 (L1188-1218): for each scheme "a reaching distance parameter
// controls the number of memory elements that Paraprox accesses ... When
// Paraprox accesses an element, its neighbors, whose distances from the
// accessed element are less than the reaching distance, will not be
// accessed"; the row/column schemes access one row/column and leave the
// rows/columns "within a reaching distance from it" unaccessed.  Readings
// S2-S5: inclusive reach, per-axis maps, centre anchor, anchors
// on a lattice of stride 2d+1, clamped to the tile edge.
//
// Because every unaccessed element is *replaced* by its representative
// (L1144-1148), the approximate output equals the filter applied to the
// substituted tile, which is the sum over representatives of (sum of the
// weights mapped to that representative) x value.  The kernels evaluate that
// folded form: |Ry|*|Rx| taps instead of K_y*K_x.
#include <algorithm>
#include <cstdlib>

#include "internal.h"

namespace ppx {

// nearest multiple of s = 2d+1 to |i| (remainder <= d rounds down, >= d+1
// rounds up; s odd -> no ties), capped at the tile radius r
int map_offset(int r, int d, int i) {
    if (d <= 0) return i;
    const int s = 2 * d + 1;
    const int a = std::abs(i);
    const int q = a / s, rem = a % s;
    int v = (rem > d ? q + 1 : q) * s;
    if (v > r) v = r;
    return i < 0 ? -v : v;
}

void scheme_reaches(paraprox_scheme s, int reach, int* dy, int* dx) {
    switch (s) {
    case PARAPROX_ROW: *dy = reach; *dx = 0; break;
    case PARAPROX_COL: *dy = 0; *dx = reach; break;
    case PARAPROX_CENTER: *dy = reach; *dx = reach; break;
    default: *dy = 0; *dx = 0; break;
    }
}

static void build_axis(int r, int d, int* m, int* reps, int* nrep, int* halo, uint32_t* mask) {
    bool used[2 * kMaxR + 1] = {};
    for (int i = -r; i <= r; ++i) {
        m[i + r] = map_offset(r, d, i);
        used[m[i + r] + kMaxR] = true;
    }
    *nrep = 0;
    *halo = 0;
    *mask = 0;
    for (int a = -kMaxR; a <= kMaxR; ++a)
        if (used[a + kMaxR]) {
            reps[(*nrep)++] = a;
            *halo = std::max(*halo, std::abs(a));
            *mask |= 1u << (a + kMaxR);
        }
}

static Plan make_plan(const paraprox_filter_s& f, int dy, int dx) {
    Plan p;
    p.ky = f.ky;
    p.kx = f.kx;
    p.ry = f.ky / 2;
    p.rx = f.kx / 2;
    p.separable = f.separable;
    p.dy = std::min(dy, p.ry);
    p.dx = std::min(dx, p.rx);
    build_axis(p.ry, p.dy, p.my, p.ay, &p.ny, &p.hy, &p.masky);
    build_axis(p.rx, p.dx, p.mx, p.ax, &p.nx, &p.hx, &p.maskx);
    auto rep_index = [](const int* reps, int n, int a) {
        for (int k = 0; k < n; ++k)
            if (reps[k] == a) return k;
        return -1;
    };
    if (f.separable) {
        double wy[kMaxK] = {}, wx[kMaxK] = {};
        for (int i = 0; i < f.ky; ++i) wy[rep_index(p.ay, p.ny, p.my[i])] += (double)f.wy[i];
        for (int j = 0; j < f.kx; ++j) wx[rep_index(p.ax, p.nx, p.mx[j])] += (double)f.wx[j];
        for (int k = 0; k < p.ny; ++k) p.wyf[k] = (float)wy[k];
        for (int k = 0; k < p.nx; ++k) p.wxf[k] = (float)wx[k];
        p.taps = p.ny + p.nx;
    } else {
        double acc[kMaxTaps] = {};
        for (int i = 0; i < f.ky; ++i)
            for (int j = 0; j < f.kx; ++j)
                acc[rep_index(p.ay, p.ny, p.my[i]) * p.nx + rep_index(p.ax, p.nx, p.mx[j])] +=
                    (double)f.w[i * f.kx + j];
        for (int k = 0; k < p.ny * p.nx; ++k) p.wf[k] = (float)acc[k];
        p.taps = p.ny * p.nx;
    }
    return p;
}

// PAPER.md §3.3.3 (L1366-1404): "Paraprox multiplies the loop step by N ...
// inserts adjustment code after the loop.  This code multiplies the result by
// the skipping rate".  Applied to the filter-row loop (rate sy) and the
// filter-column loop (rate sx): the executed offsets are -r, -r+s, ... <= r,
// and each executed weight is scaled by the rates (fp64 product, one fp32
// rounding).  Rates above the trip count K saturate to K (reading S24).
static void build_skip_axis(int r, int s, int* m, int* reps, int* nrep, int* halo, uint32_t* mask) {
    for (int i = -r; i <= r; ++i) m[i + r] = i;
    *nrep = 0;
    *halo = 0;
    *mask = 0;
    for (int a = -r; a <= r; a += s) {
        reps[(*nrep)++] = a;
        *halo = std::max(*halo, std::abs(a));
        *mask |= 1u << (a + kMaxR);
    }
}

static Plan make_plan_skip(const paraprox_filter_s& f, int sy, int sx) {
    Plan p;
    p.ky = f.ky;
    p.kx = f.kx;
    p.ry = f.ky / 2;
    p.rx = f.kx / 2;
    p.separable = f.separable;
    p.sy = std::min(sy, f.ky);
    p.sx = std::min(sx, f.kx);
    build_skip_axis(p.ry, p.sy, p.my, p.ay, &p.ny, &p.hy, &p.masky);
    build_skip_axis(p.rx, p.sx, p.mx, p.ax, &p.nx, &p.hx, &p.maskx);
    if (f.separable) {
        for (int k = 0; k < p.ny; ++k) p.wyf[k] = (float)((double)p.sy * (double)f.wy[p.ay[k] + p.ry]);
        for (int k = 0; k < p.nx; ++k) p.wxf[k] = (float)((double)p.sx * (double)f.wx[p.ax[k] + p.rx]);
        p.taps = p.ny + p.nx;
    } else {
        for (int a = 0; a < p.ny; ++a)
            for (int b = 0; b < p.nx; ++b)
                p.wf[a * p.nx + b] = (float)((double)p.sy * (double)p.sx *
                                             (double)f.w[(p.ay[a] + p.ry) * f.kx + (p.ax[b] + p.rx)]);
        p.taps = p.ny * p.nx;
    }
    return p;
}

const Plan& get_plan_skip(paraprox_filter f, int sy, int sx) {
    sy = std::min(std::max(sy, 1), f->ky);
    sx = std::min(std::max(sx, 1), f->kx);
    if (sy == 1 && sx == 1) return get_plan(f, 0, 0);
    std::lock_guard<std::mutex> lk(f->mu);
    auto key = std::make_pair(-sy, -sx);  // reach keys are >= 0
    auto it = f->plans.find(key);
    if (it == f->plans.end()) it = f->plans.emplace(key, make_plan_skip(*f, sy, sx)).first;
    return it->second;
}

bool is_skip_scheme(paraprox_scheme s) {
    return s == PARAPROX_SKIP_ROW || s == PARAPROX_SKIP_COL || s == PARAPROX_SKIP_BOTH;
}

void scheme_skips(paraprox_scheme s, int rate, int* sy, int* sx) {
    *sy = (s == PARAPROX_SKIP_ROW || s == PARAPROX_SKIP_BOTH) ? rate : 1;
    *sx = (s == PARAPROX_SKIP_COL || s == PARAPROX_SKIP_BOTH) ? rate : 1;
}

const Plan& get_plan(paraprox_filter f, int dy, int dx) {
    dy = std::min(dy, f->ky / 2);
    dx = std::min(dx, f->kx / 2);
    std::lock_guard<std::mutex> lk(f->mu);
    auto key = std::make_pair(dy, dx);
    auto it = f->plans.find(key);
    if (it == f->plans.end()) it = f->plans.emplace(key, make_plan(*f, dy, dx)).first;
    return it->second;  // std::map nodes are stable; plans are never erased
}

// Tuner candidates (reading S13): {centre, row, column} x
// reach 1..r, ordered by the integer cost key (taps, hy, hx, scheme id with
// centre < row < column, reach); a candidate whose index maps equal an
// earlier one's, or the exact maps, is dropped.
std::vector<Candidate> candidates(paraprox_filter f) {
    const int ry = f->ky / 2, rx = f->kx / 2;
    std::vector<Candidate> all;
    const paraprox_scheme order[3] = {PARAPROX_CENTER, PARAPROX_ROW, PARAPROX_COL};
    for (int s = 0; s < 3; ++s) {
        const int rmax = order[s] == PARAPROX_ROW ? ry : order[s] == PARAPROX_COL ? rx : std::max(ry, rx);
        for (int d = 1; d <= rmax; ++d) {
            Candidate c;
            c.scheme = order[s];
            c.reach = d;
            scheme_reaches(c.scheme, d, &c.dy, &c.dx);
            const Plan& p = get_plan(f, c.dy, c.dx);
            c.taps = p.taps;
            c.hy = p.hy;
            c.hx = p.hx;
            c.sid = s;
            all.push_back(c);
        }
    }
    std::stable_sort(all.begin(), all.end(), [](const Candidate& a, const Candidate& b) {
        if (a.taps != b.taps) return a.taps < b.taps;
        if (a.hy != b.hy) return a.hy < b.hy;
        if (a.hx != b.hx) return a.hx < b.hx;
        if (a.sid != b.sid) return a.sid < b.sid;
        return a.reach < b.reach;
    });
    std::vector<Candidate> out;
    const Plan& exact = get_plan(f, 0, 0);
    auto same = [&](const Plan& a, const Plan& b) {
        return std::equal(a.my, a.my + f->ky, b.my) && std::equal(a.mx, a.mx + f->kx, b.mx);
    };
    for (const Candidate& c : all) {
        const Plan& p = get_plan(f, c.dy, c.dx);
        if (same(p, exact)) continue;
        bool dup = false;
        for (const Candidate& o : out) dup = dup || same(p, get_plan(f, o.dy, o.dx));
        if (!dup) out.push_back(c);
    }
    return out;
}

}  // namespace ppx

namespace ppx {

// The extended tuner's candidates (reading S24): the stencil candidates above
// (flags bit 0) and the reduction schemes (bit 1) -- skip-both, skip-row,
// skip-col with rate N in 2..r+1 of the skipped axis (skip-both: the smaller
// radius), offered only on axes with r >= 1 -- in one order by the integer
// cost key (taps, hy, hx, scheme id: centre 0, row 1, col 2, skip-both 3,
// skip-row 4, skip-col 5, rate); a reduction candidate whose saturated rates
// equal an earlier one's is dropped.
std::vector<Candidate> candidates_ex(paraprox_filter f, int flags) {
    std::vector<Candidate> all;
    if (flags & 1) all = candidates(f);
    if (flags & 2) {
        const int ry = f->ky / 2, rx = f->kx / 2;
        const paraprox_scheme fam[3] = {PARAPROX_SKIP_BOTH, PARAPROX_SKIP_ROW, PARAPROX_SKIP_COL};
        std::vector<Candidate> sk;
        for (int q = 0; q < 3; ++q) {
            const int rmax = fam[q] == PARAPROX_SKIP_ROW ? ry : fam[q] == PARAPROX_SKIP_COL ? rx : std::min(ry, rx);
            if (rmax < 1) continue;
            for (int n = 2; n <= rmax + 1; ++n) {
                Candidate c;
                c.scheme = fam[q];
                c.reach = n;
                int sy, sx;
                scheme_skips(c.scheme, n, &sy, &sx);
                const Plan& p = get_plan_skip(f, sy, sx);
                c.dy = p.sy;  // for skip candidates dy/dx carry the saturated rates
                c.dx = p.sx;
                c.taps = p.taps;
                c.hy = p.hy;
                c.hx = p.hx;
                c.sid = 3 + q;
                bool dup = false;
                for (const Candidate& o : sk) dup = dup || (o.dy == c.dy && o.dx == c.dx);
                if (!dup) sk.push_back(c);
            }
        }
        all.insert(all.end(), sk.begin(), sk.end());
    }
    std::stable_sort(all.begin(), all.end(), [](const Candidate& a, const Candidate& b) {
        if (a.taps != b.taps) return a.taps < b.taps;
        if (a.hy != b.hy) return a.hy < b.hy;
        if (a.hx != b.hx) return a.hx < b.hx;
        if (a.sid != b.sid) return a.sid < b.sid;
        return a.reach < b.reach;
    });
    return all;
}

}  // namespace ppx
