// Host algorithms: FPM evaluation, geometric FPM partitioning, column-based
// arrangement and pivot delivery plan.  Compiled with -ffp-contract=off and
// without fast-math so the floating-point results are bit-identical to the
// specification in DESIGN.md (readings Q1-Q4, Q10, Q12).
#include "host_algos.hpp"

#include <algorithm>
#include <cmath>
#include <tuple>

#include "../common.hpp"

namespace fpm {

// ---------------------------------------------------------------- models
void validate_model(const fpm_model& m, int idx) {
    FPM_CHECK_ARG(m.npts >= 1 && m.x && m.s, "model %d: npts must be >= 1 with non-null x, s", idx);
    for (int j = 0; j < m.npts; ++j) {
        FPM_CHECK_ARG(m.x[j] >= 1, "model %d: x[%d] = %lld < 1", idx, j, (long long)m.x[j]);
        FPM_CHECK_ARG(j == 0 || m.x[j] > m.x[j - 1], "model %d: x not strictly increasing at %d", idx, j);
        FPM_CHECK_ARG(std::isfinite(m.s[j]) && m.s[j] > 0.0, "model %d: s[%d] must be finite and > 0",
                      idx, j);
    }
}

// s(x): P:8 "represents the processor speed by a function of problem size".
// Piecewise linear between sample points, constant beyond the ends (Q4).  The
// expression order is part of the specification.
double model_speed(const fpm_model& m, int64_t x) {
    const int L = m.npts - 1;
    if (x <= m.x[0]) return m.s[0];
    if (x >= m.x[L]) return m.s[L];
    int lo = 0, hi = L;  // invariant: x[lo] <= x < x[hi]
    while (hi - lo > 1) {
        const int mid = (lo + hi) / 2;
        if (m.x[mid] <= x) lo = mid; else hi = mid;
    }
    return m.s[lo] + (m.s[lo + 1] - m.s[lo]) * (double)(x - m.x[lo]) / (double)(m.x[lo + 1] - m.x[lo]);
}

double model_time(const fpm_model& m, int64_t x) {
    if (x == 0) return 0.0;
    return (double)x / model_speed(m, x);
}

// ------------------------------------------------------ continuous geometry
// Speed at a real problem size (same piecewise-linear model).
static double speed_real(const fpm_model& m, double x) {
    const int L = m.npts - 1;
    if (x <= (double)m.x[0]) return m.s[0];
    if (x >= (double)m.x[L]) return m.s[L];
    int j = 0;
    while ((double)m.x[j + 1] <= x) ++j;
    return m.s[j] + (m.s[j + 1] - m.s[j]) * (x - (double)m.x[j]) / (double)(m.x[j + 1] - m.x[j]);
}

// x_i(tau): the largest real x whose time x / s(x) is <= tau, i.e. where the
// line through the origin y = x / tau leaves the speed graph ([5]).  On
// every linear piece t(x) is monotone, so each piece is solved in closed form.
static double reach(const fpm_model& m, double tau) {
    const int L = m.npts - 1;
    if (tau * m.s[L] >= (double)m.x[L]) return tau * m.s[L];
    for (int j = L - 1; j >= 0; --j) {
        const double x0 = (double)m.x[j], x1 = (double)m.x[j + 1];
        const double t0 = x0 / m.s[j], t1 = x1 / m.s[j + 1];
        if (t1 <= tau) return x1;
        if (t0 <= tau) {
            const double c = (m.s[j + 1] - m.s[j]) / (x1 - x0);
            const double a = m.s[j] - c * x0;
            const double den = 1.0 - tau * c;
            if (!(den > 0.0)) return x0;
            return std::min(std::max(tau * a / den, x0), x1);
        }
    }
    return std::min(tau * m.s[0], (double)m.x[0]);
}

// ---------------------------------------------------------------- partition
namespace {
// Prefix maxima m_i(j) = max_{l <= j} t_i(l), filled on demand.
struct PrefixTimes {
    const fpm_model* m;
    std::vector<double> pm{0.0};  // pm[0] = t(0) = 0
    double at(int64_t j) {
        while ((int64_t)pm.size() <= j) {
            const int64_t l = (int64_t)pm.size();
            pm.push_back(std::max(pm.back(), model_time(*m, l)));
        }
        return pm[j];
    }
};
using Key = std::tuple<double, int, int64_t>;  // (m_i(j), i, j)
}  // namespace

// FPM-based partitioning: P:9 equal completion time; P:15 areas "proportional to
// the speed of the processor ... given by the speed function ... for the
// assigned problem size"; the algorithm is that of [5]:
//  (1) geometric phase: bisection of the line through the origin (here on its
//      inverse slope tau = time) between bounds from the even share T/p, until
//      every floor(x_i) agrees at both ends (or 200 iterations);
//  (2) exact integer phase on the keys (m_i(j), i, j), m_i = prefix maxima of
//      t_i: adjust sum d to T, then exchange the largest included key with the
//      smallest excluded one until none is larger.  The T smallest such keys are
//      exactly what giving blocks one by one to the device with the smallest
//      t_i(d_i + 1) produces, so the output
//      is the canonical partition, bit for bit.
int partition(int64_t T, int p, const fpm_model* models, int64_t* d_out) {
    FPM_CHECK_ARG(p >= 1 && p <= FPM_MAX_DEVICES, "p = %d out of [1, %d]", p, FPM_MAX_DEVICES);
    FPM_CHECK_ARG(T >= 0, "total_blocks < 0");
    for (int i = 0; i < p; ++i) validate_model(models[i], i);
    for (int i = 0; i < p; ++i) d_out[i] = 0;
    if (T == 0) return 0;
    if (p == 1) {
        d_out[0] = T;
        return 0;
    }

    // (1) geometric bisection.
    const double share = (double)T / (double)p;
    double tau_lo = 0.0, tau_hi = 0.0;
    for (int i = 0; i < p; ++i) {
        const double t = share / speed_real(models[i], share);
        tau_lo = (i == 0) ? t : std::min(tau_lo, t);
        tau_hi = (i == 0) ? t : std::max(tau_hi, t);
    }
    auto total = [&](double tau) {
        double s = 0.0;
        for (int i = 0; i < p; ++i) s += reach(models[i], tau);
        return s;
    };
    for (int g = 0; g < 64 && total(tau_lo) > (double)T; ++g) tau_lo *= 0.5;
    for (int g = 0; g < 64 && total(tau_hi) < (double)T; ++g) tau_hi *= 2.0;
    int iters = 0;
    for (; iters < 200; ++iters) {
        bool same = true;
        for (int i = 0; i < p && same; ++i)
            same = std::floor(reach(models[i], tau_lo)) == std::floor(reach(models[i], tau_hi));
        if (same) break;
        const double mid = 0.5 * (tau_lo + tau_hi);
        if (!(mid > tau_lo && mid < tau_hi)) break;
        if (total(mid) <= (double)T) tau_lo = mid; else tau_hi = mid;
    }
    std::vector<int64_t> d(p);
    for (int i = 0; i < p; ++i) {
        const double x = std::floor(reach(models[i], tau_lo));
        d[i] = (int64_t)std::min(std::max(x, 0.0), (double)T);
    }

    // (2) exact integer phase.
    std::vector<PrefixTimes> pt(p);
    for (int i = 0; i < p; ++i) pt[i].m = &models[i];
    auto inc_key = [&](int i) { return Key(pt[i].at(d[i]), i, d[i]); };
    auto fr_key = [&](int i) { return Key(pt[i].at(d[i] + 1), i, d[i] + 1); };
    auto argmax_inc = [&]() {
        int best = -1;
        for (int i = 0; i < p; ++i)
            if (d[i] > 0 && (best < 0 || inc_key(i) > inc_key(best))) best = i;
        return best;
    };
    auto argmin_fr = [&]() {
        int best = 0;
        for (int i = 1; i < p; ++i)
            if (fr_key(i) < fr_key(best)) best = i;
        return best;
    };
    int64_t sum = 0;
    for (int i = 0; i < p; ++i) sum += d[i];
    while (sum > T) { --d[argmax_inc()]; --sum; }
    while (sum < T) { ++d[argmin_fr()]; ++sum; }
    for (;;) {
        const int a = argmax_inc(), b = argmin_fr();
        if (a < 0 || !(inc_key(a) > fr_key(b))) break;
        --d[a];
        ++d[b];
    }
    for (int i = 0; i < p; ++i) d_out[i] = d[i];
    return iters;
}

// ---------------------------------------------------------------- arrangement
static std::vector<int64_t> largest_remainder(const std::vector<int64_t>& num, int64_t den,
                                              int64_t total) {
    const size_t k = num.size();
    std::vector<int64_t> out(k), rem(k);
    int64_t s = 0;
    for (size_t i = 0; i < k; ++i) {
        out[i] = num[i] / den;
        rem[i] = num[i] % den;
        s += out[i];
    }
    std::vector<size_t> idx(k);
    for (size_t i = 0; i < k; ++i) idx[i] = i;
    std::stable_sort(idx.begin(), idx.end(), [&](size_t a, size_t b) { return rem[a] > rem[b]; });
    for (int64_t l = 0; l < total - s; ++l) out[idx[(size_t)l]] += 1;
    return out;
}

// Column-based arrangement: rectangles of areas ~ d_i "as square as
// possible, minimising the total volume of communications" ([17], reading Q10):
// sort by (-d_i, i), best split into consecutive columns by
// (sum_j k_j A_j + T, #columns, column sizes), largest-remainder widths/heights.
void arrange(int64_t n, int p, const int64_t* d, colpart_rect* out) {
    FPM_CHECK_ARG(n >= 1, "n must be >= 1");
    FPM_CHECK_ARG(p >= 1 && p <= FPM_MAX_DEVICES, "p = %d out of [1, %d]", p, FPM_MAX_DEVICES);
    const int64_t T = n * n;
    int64_t sum = 0;
    for (int i = 0; i < p; ++i) {
        FPM_CHECK_ARG(d[i] >= 0, "d[%d] < 0", i);
        sum += d[i];
    }
    FPM_CHECK_ARG(sum == T, "sum of areas %lld != n*n = %lld", (long long)sum, (long long)T);

    std::vector<int> order(p);
    for (int i = 0; i < p; ++i) order[i] = i;
    std::sort(order.begin(), order.end(), [&](int a, int b) {
        return d[a] != d[b] ? d[a] > d[b] : a < b;
    });
    std::vector<int> active;
    for (int i : order)
        if (d[i] > 0) active.push_back(i);
    const int q = (int)active.size();

    // best split of `active` into consecutive groups
    uint32_t best_mask = 0;
    int64_t best_cost = -1;
    int best_cols = 0;
    std::vector<int> best_sizes;
    for (uint32_t mask = 0; mask < (1u << (q - 1)); ++mask) {
        int64_t cost = 0, area = 0;
        int cols = 0, cnt = 0;
        std::vector<int> sizes;
        for (int pos = 0; pos < q; ++pos) {
            if (pos > 0 && (mask & (1u << (pos - 1)))) {
                cost += cnt * area + T;
                sizes.push_back(cnt);
                ++cols;
                area = 0;
                cnt = 0;
            }
            area += d[active[pos]];
            ++cnt;
        }
        cost += cnt * area + T;
        sizes.push_back(cnt);
        ++cols;
        const bool better = best_cost < 0 || cost < best_cost ||
                            (cost == best_cost && (cols < best_cols ||
                                                   (cols == best_cols && sizes < best_sizes)));
        if (better) {
            best_cost = cost;
            best_cols = cols;
            best_sizes = sizes;
            best_mask = mask;
        }
    }

    std::vector<std::vector<int>> groups(1);
    for (int pos = 0; pos < q; ++pos) {
        if (pos > 0 && (best_mask & (1u << (pos - 1)))) groups.emplace_back();
        groups.back().push_back(active[pos]);
    }
    std::vector<int64_t> areas;
    for (auto& g : groups) {
        int64_t a = 0;
        for (int i : g) a += d[i];
        areas.push_back(a);
    }
    const std::vector<int64_t> widths = largest_remainder(areas, n, n);
    for (int i = 0; i < p; ++i) out[i] = colpart_rect{-1, 0, 0, 0, 0};
    int64_t col0 = 0;
    for (size_t j = 0; j < groups.size(); ++j) {
        std::vector<int64_t> num;
        for (int i : groups[j]) num.push_back(n * d[i]);
        const std::vector<int64_t> heights = largest_remainder(num, areas[j], n);
        int64_t row0 = 0;
        for (size_t k = 0; k < groups[j].size(); ++k) {
            out[groups[j][k]] = colpart_rect{(int32_t)j, row0, col0, heights[k], widths[j]};
            row0 += heights[k];
        }
        col0 += widths[j];
    }
}

// FPM-chosen integers for the column-based arrangement (reading Q25, SURVEY
// NEXT-4): every consecutive split of the (-d_i, i) order into columns; per
// column and width w the heights come from the equal-time greedy on the rows
// (P:9), the widths from the same greedy on the columns; the split with the
// least (makespan, half-perimeter sum, #columns, column sizes) wins.
// Column times are memoised per (first device, devices, width): O(q^3 n^2 / 6)
// model evaluations for q live devices.
void arrange_fpm(int64_t n, int p, const int64_t* d, const fpm_model* models, colpart_rect* out) {
    FPM_CHECK_ARG(n >= 1 && n <= 1024, "n = %lld out of [1, 1024] for the FPM arrangement", (long long)n);
    FPM_CHECK_ARG(p >= 1 && p <= FPM_MAX_DEVICES, "p = %d out of [1, %d]", p, FPM_MAX_DEVICES);
    int64_t sum = 0;
    for (int i = 0; i < p; ++i) {
        FPM_CHECK_ARG(d[i] >= 0, "d[%d] < 0", i);
        sum += d[i];
        validate_model(models[i], i);
    }
    FPM_CHECK_ARG(sum == n * n, "sum of areas %lld != n*n = %lld", (long long)sum, (long long)(n * n));

    std::vector<int> order(p);
    for (int i = 0; i < p; ++i) order[i] = i;
    std::sort(order.begin(), order.end(), [&](int a, int b) { return d[a] != d[b] ? d[a] > d[b] : a < b; });
    std::vector<int> active;
    for (int i : order)
        if (d[i] > 0) active.push_back(i);
    const int q = (int)active.size();

    // heights of the column active[start .. start+len) at width w (rows from zero,
    // one at a time to the least (t((h+1) w), position)); returns the column time
    auto heights = [&](int start, int len, int64_t w, std::vector<int64_t>& h) {
        h.assign(len, 0);
        for (int64_t r = 0; r < n; ++r) {
            int best = -1;
            double bt = 0.0;
            for (int m = 0; m < len; ++m) {
                const double t = model_time(models[active[start + m]], (h[m] + 1) * w);
                if (best < 0 || t < bt) {
                    best = m;
                    bt = t;
                }
            }
            ++h[best];
        }
        double mx = 0.0;
        for (int m = 0; m < len; ++m) mx = std::max(mx, model_time(models[active[start + m]], h[m] * w));
        return mx;
    };
    std::vector<double> memo((size_t)q * q * (n + 1), -1.0);
    std::vector<int64_t> scratch;
    auto col_time = [&](int start, int len, int64_t w) {
        double& v = memo[((size_t)start * q + (len - 1)) * (n + 1) + w];
        if (v < 0.0) v = heights(start, len, w, scratch);
        return v;
    };

    bool have = false;
    double best_ms = 0.0;
    int64_t best_cost = 0;
    std::vector<int> best_sizes, best_starts;
    std::vector<int64_t> best_w;
    for (uint32_t mask = 0; mask < (1u << (q - 1)); ++mask) {
        std::vector<int> starts{0}, sizes;
        for (int pos = 1; pos < q; ++pos)
            if (mask & (1u << (pos - 1))) starts.push_back(pos);
        for (size_t j = 0; j < starts.size(); ++j)
            sizes.push_back((j + 1 < starts.size() ? starts[j + 1] : q) - starts[j]);
        const int c = (int)starts.size();
        std::vector<int64_t> w(c, 0);
        for (int64_t step = 0; step < n; ++step) {
            int bj = -1;
            double bt = 0.0;
            for (int j = 0; j < c; ++j) {
                const double t = col_time(starts[j], sizes[j], w[j] + 1);
                if (bj < 0 || t < bt) {
                    bj = j;
                    bt = t;
                }
            }
            ++w[bj];
        }
        double ms = 0.0;
        int64_t cost = 0;
        for (int j = 0; j < c; ++j) {
            ms = std::max(ms, col_time(starts[j], sizes[j], w[j]));
            heights(starts[j], sizes[j], w[j], scratch);
            for (int64_t h : scratch)
                if (h * w[j] > 0) cost += h + w[j];
        }
        const bool better = !have || ms < best_ms ||
                            (ms == best_ms && (cost < best_cost ||
                                               (cost == best_cost && (c < (int)best_sizes.size() ||
                                                                      (c == (int)best_sizes.size() &&
                                                                       sizes < best_sizes)))));
        if (better) {
            have = true;
            best_ms = ms;
            best_cost = cost;
            best_sizes = sizes;
            best_starts = starts;
            best_w = w;
        }
    }

    for (int i = 0; i < p; ++i) out[i] = colpart_rect{-1, 0, 0, 0, 0};
    int64_t col0 = 0;
    int32_t col = 0;
    for (size_t j = 0; j < best_starts.size(); ++j) {
        if (best_w[j] == 0) continue;
        std::vector<int64_t> h;
        heights(best_starts[j], best_sizes[j], best_w[j], h);
        int64_t row0 = 0;
        for (int m = 0; m < best_sizes[j]; ++m) {
            if (h[m] > 0) out[active[best_starts[j] + m]] = colpart_rect{col, row0, col0, h[m], best_w[j]};
            row0 += h[m];
        }
        col0 += best_w[j];
        ++col;
    }
}

void validate_rects(int64_t n, int p, const colpart_rect* r) {
    FPM_CHECK_ARG(n >= 1 && p >= 1 && p <= FPM_MAX_DEVICES, "bad n or p");
    // columns: same col0/w for all live members; widths partition [0, n); rows
    // of each column partition [0, n).
    struct Col { int64_t col0 = -1, w = -1; std::vector<std::pair<int64_t, int64_t>> rows; };
    std::vector<Col> cols;
    for (int i = 0; i < p; ++i) {
        FPM_CHECK_ARG(r[i].h >= 0 && r[i].w >= 0 && r[i].row0 >= 0 && r[i].col0 >= 0,
                      "rect %d has negative fields", i);
        if (r[i].h == 0 || r[i].w == 0) continue;
        FPM_CHECK_ARG(r[i].col >= 0 && r[i].col < FPM_MAX_DEVICES, "rect %d: bad column id", i);
        if ((int)cols.size() <= r[i].col) cols.resize(r[i].col + 1);
        Col& c = cols[r[i].col];
        if (c.w < 0) { c.col0 = r[i].col0; c.w = r[i].w; }
        FPM_CHECK_ARG(c.col0 == r[i].col0 && c.w == r[i].w, "rect %d: column %d inconsistent", i, r[i].col);
        c.rows.push_back({r[i].row0, r[i].h});
    }
    std::vector<std::pair<int64_t, int64_t>> spans;
    for (auto& c : cols) {
        if (c.w < 0) continue;
        spans.push_back({c.col0, c.w});
        std::sort(c.rows.begin(), c.rows.end());
        int64_t at = 0;
        for (auto& rw : c.rows) {
            FPM_CHECK_ARG(rw.first == at, "column rows do not tile [0, n)");
            at += rw.second;
        }
        FPM_CHECK_ARG(at == n, "column rows do not tile [0, n)");
    }
    std::sort(spans.begin(), spans.end());
    int64_t at = 0;
    for (auto& s : spans) {
        FPM_CHECK_ARG(s.first == at, "columns do not tile [0, n)");
        at += s.second;
    }
    FPM_CHECK_ARG(at == n, "columns do not tile [0, n)");
}

// Iteration k: the devices of the column holding block-column k send
// A(rows, k) to every device whose rows overlap theirs; in every column the
// device whose rows hold block-row k sends B(k, cols) to its column (Q12).
void plan_step(int64_t n, int p, const colpart_rect* r, int64_t k, std::vector<Move>& am,
               std::vector<Move>& bm) {
    FPM_CHECK_ARG(k >= 0 && k < n, "k out of range");
    am.clear();
    bm.clear();
    auto live = [&](int i) { return r[i].h > 0 && r[i].w > 0; };
    for (int i = 0; i < p; ++i) {
        if (!live(i)) continue;
        for (int q = 0; q < p; ++q) {
            if (!live(q) || !(r[q].col0 <= k && k < r[q].col0 + r[q].w)) continue;
            const int64_t lo = std::max(r[i].row0, r[q].row0);
            const int64_t hi = std::min(r[i].row0 + r[i].h, r[q].row0 + r[q].h);
            if (lo < hi) am.push_back(Move{q, i, lo, hi});
        }
        int owner = -1;
        for (int q = 0; q < p; ++q)
            if (live(q) && r[q].col == r[i].col && r[q].row0 <= k && k < r[q].row0 + r[q].h) owner = q;
        FPM_CHECK_ARG(owner >= 0, "no owner of block-row %lld in column %d", (long long)k, r[i].col);
        bm.push_back(Move{owner, i, r[i].col0, r[i].col0 + r[i].w});
    }
    auto lt = [](const Move& a, const Move& b) {
        return std::tie(a.src, a.dst, a.begin, a.end) < std::tie(b.src, b.dst, b.begin, b.end);
    };
    std::sort(am.begin(), am.end(), lt);
    std::sort(bm.begin(), bm.end(), lt);
}

}  // namespace fpm

// ------------------------------------------------------------------- C ABI
extern "C" int fpm_model_speed(const fpm_model* model, int64_t x, double* s_out) {
    return fpm::guarded([&] {
        FPM_CHECK_ARG(model && s_out, "null argument");
        FPM_CHECK_ARG(x >= 0, "x < 0");
        fpm::validate_model(*model, 0);
        *s_out = fpm::model_speed(*model, x);
    });
}

extern "C" int fpm_partition(int64_t total_blocks, int32_t p, const fpm_model* models, int64_t* d_out,
                             int32_t* iters_out) {
    return fpm::guarded([&] {
        FPM_CHECK_ARG(models && d_out, "null argument");
        const int it = fpm::partition(total_blocks, p, models, d_out);
        if (iters_out) *iters_out = it;
    });
}

extern "C" int colpart_arrange(int64_t n, int32_t p, const int64_t* d, colpart_rect* rects_out) {
    return fpm::guarded([&] {
        FPM_CHECK_ARG(d && rects_out, "null argument");
        fpm::arrange(n, p, d, rects_out);
    });
}

extern "C" int colpart_arrange_fpm(int64_t n, int32_t p, const int64_t* d, const fpm_model* models,
                                  colpart_rect* rects_out) {
    return fpm::guarded([&] {
        FPM_CHECK_ARG(d && models && rects_out, "null argument");
        fpm::arrange_fpm(n, p, d, models, rects_out);
    });
}

extern "C" int colpart_plan_step(int64_t n, int32_t p, const colpart_rect* rects, int64_t k,
                                 colpart_move* a_moves, int32_t a_cap, int32_t* a_count,
                                 colpart_move* b_moves, int32_t b_cap, int32_t* b_count) {
    return fpm::guarded([&] {
        FPM_CHECK_ARG(rects && a_count && b_count, "null argument");
        fpm::validate_rects(n, p, rects);
        std::vector<fpm::Move> am, bm;
        fpm::plan_step(n, p, rects, k, am, bm);
        *a_count = (int32_t)am.size();
        *b_count = (int32_t)bm.size();
        FPM_CHECK_ARG((int32_t)am.size() <= a_cap && (int32_t)bm.size() <= b_cap,
                      "move capacity too small (need %zu A, %zu B)", am.size(), bm.size());
        for (size_t i = 0; i < am.size(); ++i)
            a_moves[i] = colpart_move{am[i].src, am[i].dst, am[i].begin, am[i].end};
        for (size_t i = 0; i < bm.size(); ++i)
            b_moves[i] = colpart_move{bm[i].src, bm[i].dst, bm[i].begin, bm[i].end};
    });
}
