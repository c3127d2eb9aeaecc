// Host-side algorithms of the method (pure C++, no CUDA): model evaluation,
// FPM partitioning, column-based arrangement, pivot delivery plan.
#pragma once

#include <cstdint>
#include <vector>

#include "fpmpmm.h"

namespace fpm {

void validate_model(const fpm_model& m, int idx);
double model_speed(const fpm_model& m, int64_t x);  // P:8, reading Q4
double model_time(const fpm_model& m, int64_t x);   // x / s(x), t(0) = 0

// FPM partition (P:9, [5] P:129).  Returns bisection iterations.
int partition(int64_t T, int p, const fpm_model* models, int64_t* d_out);

// Column-based arrangement ([17] P:144).
void arrange(int64_t n, int p, const int64_t* d, colpart_rect* out);

// Column-based arrangement with FPM-chosen integer widths / heights (Q25).
void arrange_fpm(int64_t n, int p, const int64_t* d, const fpm_model* models, colpart_rect* out);

// Checks that rects form a column-based tiling of the n x n grid.
void validate_rects(int64_t n, int p, const colpart_rect* rects);

struct Move {
    int32_t src, dst;
    int64_t begin, end;
};
// Pivot delivery of iteration k (reading Q12), sorted by (src, dst, begin).
void plan_step(int64_t n, int p, const colpart_rect* rects, int64_t k, std::vector<Move>& a_moves,
               std::vector<Move>& b_moves);

}  // namespace fpm
