// Host-CPU devices: pinned worker teams and the product-side GEMM they run
// (cpu_device.hpp; PAPER.md P:10-11, P:18 -- the paper's sockets run the ACML
// GEMM on all their cores at once).
//
// GEMM structure (Goto / BLIS blocking, row-major):
//   for jc in N by NC:  for pc in K by KC:
//     pack B(pc.., jc..) into NR-column micro-panels  (all threads share the work)
//     barrier
//     for ic in this thread's rows by MC:
//       pack A(ic.., pc..) into MR-row micro-panels    (per thread)
//       for jr over the NR panels:  for ir over the MR panels:
//         micro-kernel: MR x NR tile of C += A~ B~ over KC (registers), then
//         C = (first K-block and !accumulate ? 0 : C) + tile
//     barrier
// Micro-kernels: AVX-512 12 x 32 (FP32) / 12 x 16 (FP64), 24 zmm accumulators;
// AVX2 6 x 16 / 6 x 8, 12 ymm accumulators; chosen at run time (cpuid).
#include "cpu_device.hpp"

#include <immintrin.h>
#include <pthread.h>
#include <sched.h>

#include <algorithm>
#include <atomic>
#include <condition_variable>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <memory>
#include <mutex>
#include <thread>

#include "../common.hpp"

namespace fpm {
namespace cpu {

// ------------------------------------------------------------------ team
struct Team {
    std::vector<std::thread> workers;
    std::mutex mu;
    std::condition_variable cv, cv_done;
    std::function<void(int, int)> job;
    uint64_t generation = 0;
    int running = 0;
    bool stop = false;
    // spin barrier used inside a job
    std::atomic<int> bar_count{0};
    std::atomic<int> bar_sense{0};
    int n = 1;
    // packing buffers (one B buffer shared, one A buffer per thread), grown on demand
    std::vector<void*> a_buf;
    std::vector<size_t> a_cap;
    void* b_buf = nullptr;
    size_t b_cap = 0;

    void barrier() {
        const int s = bar_sense.load(std::memory_order_relaxed);
        if (bar_count.fetch_add(1, std::memory_order_acq_rel) == n - 1) {
            bar_count.store(0, std::memory_order_relaxed);
            bar_sense.store(s ^ 1, std::memory_order_release);
        } else {
            while (bar_sense.load(std::memory_order_acquire) == s) _mm_pause();
        }
    }

    // Run fn(tid, n) on every worker; returns when all finished.
    void run(const std::function<void(int, int)>& fn) {
        {
            std::unique_lock<std::mutex> lk(mu);
            job = fn;
            running = n;
            ++generation;
        }
        cv.notify_all();
        std::unique_lock<std::mutex> lk(mu);
        cv_done.wait(lk, [&] { return running == 0; });
        job = nullptr;
    }
};

namespace {

void worker_main(Team* t, int tid, int core) {
    if (core >= 0) {
        cpu_set_t set;
        CPU_ZERO(&set);
        CPU_SET(core, &set);
        pthread_setaffinity_np(pthread_self(), sizeof(set), &set);  // P:10 (i): processes bound to cores
    }
    uint64_t seen = 0;
    for (;;) {
        std::function<void(int, int)> fn;
        {
            std::unique_lock<std::mutex> lk(t->mu);
            t->cv.wait(lk, [&] { return t->stop || t->generation != seen; });
            if (t->stop) return;
            seen = t->generation;
            fn = t->job;
        }
        fn(tid, t->n);
        {
            std::lock_guard<std::mutex> lk(t->mu);
            if (--t->running == 0) t->cv_done.notify_all();
        }
    }
}

void* aligned(size_t bytes) {
    void* p = nullptr;
    if (posix_memalign(&p, 64, std::max<size_t>(bytes, 64)) != 0) throw std::bad_alloc();
    return p;
}

}  // namespace

std::vector<int> allowed_cores() {
    cpu_set_t set;
    CPU_ZERO(&set);
    std::vector<int> out;
    if (sched_getaffinity(0, sizeof(set), &set) == 0) {
        for (int c = 0; c < CPU_SETSIZE; ++c)
            if (CPU_ISSET(c, &set)) out.push_back(c);
    }
    if (out.empty()) {
        const unsigned hc = std::max(1u, std::thread::hardware_concurrency());
        for (unsigned c = 0; c < hc; ++c) out.push_back((int)c);
    }
    return out;
}

Team* team_create(const std::vector<int>& cores, int n) {
    auto t = std::make_unique<Team>();
    t->n = cores.empty() ? std::max(1, n) : (int)cores.size();
    t->a_buf.assign(t->n, nullptr);
    t->a_cap.assign(t->n, 0);
    for (int i = 0; i < t->n; ++i) t->workers.emplace_back(worker_main, t.get(), i, cores.empty() ? -1 : cores[i]);
    return t.release();
}

void team_destroy(Team* t) {
    if (!t) return;
    {
        std::lock_guard<std::mutex> lk(t->mu);
        t->stop = true;
    }
    t->cv.notify_all();
    for (auto& w : t->workers) w.join();
    for (void* p : t->a_buf) std::free(p);
    std::free(t->b_buf);
    delete t;
}

// ------------------------------------------------------------------ micro-kernels
namespace {

bool have_avx512() {
    static const bool v = __builtin_cpu_supports("avx512f") != 0;
    return v;
}
bool have_avx2() {
    static const bool v = __builtin_cpu_supports("avx2") != 0 && __builtin_cpu_supports("fma") != 0;
    return v;
}

// c (MR x NR, ldc) = (load_c ? c : 0) + sum_k a[k][0..MR) (x) b[k][0..NR)
__attribute__((target("avx512f"))) void uk_f32_512(int64_t kc, const float* __restrict a, const float* __restrict b,
                                                     float* __restrict c, int64_t ldc, bool load_c) {
    __m512 x0[12], x1[12];
#pragma GCC unroll 12
    for (int i = 0; i < 12; ++i) x0[i] = x1[i] = _mm512_setzero_ps();
    for (int64_t k = 0; k < kc; ++k) {
        const __m512 b0 = _mm512_load_ps(b), b1 = _mm512_load_ps(b + 16);
#pragma GCC unroll 12
        for (int i = 0; i < 12; ++i) {
            const __m512 ai = _mm512_set1_ps(a[i]);
            x0[i] = _mm512_fmadd_ps(ai, b0, x0[i]);
            x1[i] = _mm512_fmadd_ps(ai, b1, x1[i]);
        }
        a += 12;
        b += 32;
    }
#pragma GCC unroll 12
    for (int i = 0; i < 12; ++i) {
        float* ci = c + i * ldc;
        if (load_c) {
            x0[i] = _mm512_add_ps(_mm512_loadu_ps(ci), x0[i]);
            x1[i] = _mm512_add_ps(_mm512_loadu_ps(ci + 16), x1[i]);
        }
        _mm512_storeu_ps(ci, x0[i]);
        _mm512_storeu_ps(ci + 16, x1[i]);
    }
}

__attribute__((target("avx512f"))) void uk_f64_512(int64_t kc, const double* __restrict a, const double* __restrict b,
                                                     double* __restrict c, int64_t ldc, bool load_c) {
    __m512d x0[12], x1[12];
#pragma GCC unroll 12
    for (int i = 0; i < 12; ++i) x0[i] = x1[i] = _mm512_setzero_pd();
    for (int64_t k = 0; k < kc; ++k) {
        const __m512d b0 = _mm512_load_pd(b), b1 = _mm512_load_pd(b + 8);
#pragma GCC unroll 12
        for (int i = 0; i < 12; ++i) {
            const __m512d ai = _mm512_set1_pd(a[i]);
            x0[i] = _mm512_fmadd_pd(ai, b0, x0[i]);
            x1[i] = _mm512_fmadd_pd(ai, b1, x1[i]);
        }
        a += 12;
        b += 16;
    }
#pragma GCC unroll 12
    for (int i = 0; i < 12; ++i) {
        double* ci = c + i * ldc;
        if (load_c) {
            x0[i] = _mm512_add_pd(_mm512_loadu_pd(ci), x0[i]);
            x1[i] = _mm512_add_pd(_mm512_loadu_pd(ci + 8), x1[i]);
        }
        _mm512_storeu_pd(ci, x0[i]);
        _mm512_storeu_pd(ci + 8, x1[i]);
    }
}

__attribute__((target("avx2,fma"))) void uk_f32_256(int64_t kc, const float* __restrict a, const float* __restrict b,
                                                      float* __restrict c, int64_t ldc, bool load_c) {
    __m256 x0[6], x1[6];
#pragma GCC unroll 6
    for (int i = 0; i < 6; ++i) x0[i] = x1[i] = _mm256_setzero_ps();
    for (int64_t k = 0; k < kc; ++k) {
        const __m256 b0 = _mm256_load_ps(b), b1 = _mm256_load_ps(b + 8);
#pragma GCC unroll 6
        for (int i = 0; i < 6; ++i) {
            const __m256 ai = _mm256_broadcast_ss(a + i);
            x0[i] = _mm256_fmadd_ps(ai, b0, x0[i]);
            x1[i] = _mm256_fmadd_ps(ai, b1, x1[i]);
        }
        a += 6;
        b += 16;
    }
#pragma GCC unroll 6
    for (int i = 0; i < 6; ++i) {
        float* ci = c + i * ldc;
        if (load_c) {
            x0[i] = _mm256_add_ps(_mm256_loadu_ps(ci), x0[i]);
            x1[i] = _mm256_add_ps(_mm256_loadu_ps(ci + 8), x1[i]);
        }
        _mm256_storeu_ps(ci, x0[i]);
        _mm256_storeu_ps(ci + 8, x1[i]);
    }
}

__attribute__((target("avx2,fma"))) void uk_f64_256(int64_t kc, const double* __restrict a, const double* __restrict b,
                                                      double* __restrict c, int64_t ldc, bool load_c) {
    __m256d x0[6], x1[6];
#pragma GCC unroll 6
    for (int i = 0; i < 6; ++i) x0[i] = x1[i] = _mm256_setzero_pd();
    for (int64_t k = 0; k < kc; ++k) {
        const __m256d b0 = _mm256_load_pd(b), b1 = _mm256_load_pd(b + 4);
#pragma GCC unroll 6
        for (int i = 0; i < 6; ++i) {
            const __m256d ai = _mm256_broadcast_sd(a + i);
            x0[i] = _mm256_fmadd_pd(ai, b0, x0[i]);
            x1[i] = _mm256_fmadd_pd(ai, b1, x1[i]);
        }
        a += 6;
        b += 8;
    }
#pragma GCC unroll 6
    for (int i = 0; i < 6; ++i) {
        double* ci = c + i * ldc;
        if (load_c) {
            x0[i] = _mm256_add_pd(_mm256_loadu_pd(ci), x0[i]);
            x1[i] = _mm256_add_pd(_mm256_loadu_pd(ci + 4), x1[i]);
        }
        _mm256_storeu_pd(ci, x0[i]);
        _mm256_storeu_pd(ci + 4, x1[i]);
    }
}

// Portable micro-kernel (4 x 8): machines without AVX2.  std::fma keeps the
// arithmetic the same as the vector kernels (one rounding per multiply-add).
template <class T>
void uk_generic(int64_t kc, const T* __restrict a, const T* __restrict b, T* __restrict c, int64_t ldc, bool load_c) {
    T x[4][8] = {};
    for (int64_t k = 0; k < kc; ++k) {
        for (int i = 0; i < 4; ++i)
            for (int j = 0; j < 8; ++j) x[i][j] = std::fma(a[i], b[j], x[i][j]);
        a += 4;
        b += 8;
    }
    for (int i = 0; i < 4; ++i)
        for (int j = 0; j < 8; ++j) c[i * ldc + j] = load_c ? c[i * ldc + j] + x[i][j] : x[i][j];
}

template <class T>
struct Kernel {
    int MR, NR;
    void (*uk)(int64_t, const T*, const T*, T*, int64_t, bool);
};

template <class T>
Kernel<T> pick();
template <>
Kernel<float> pick<float>() {
    if (have_avx512()) return {12, 32, uk_f32_512};
    if (have_avx2()) return {6, 16, uk_f32_256};
    return {4, 8, uk_generic<float>};
}
template <>
Kernel<double> pick<double>() {
    if (have_avx512()) return {12, 16, uk_f64_512};
    if (have_avx2()) return {6, 8, uk_f64_256};
    return {4, 8, uk_generic<double>};
}

constexpr int64_t KC = 256;   // K block: an NR x KC B micro-panel stays in L1 (32 KB FP32)
constexpr int64_t MC = 96;    // rows per packed A block (L2)
constexpr int64_t NC = 3072;  // columns per packed B block (shared, L3)

template <class T>
void gemm(Team* t, int64_t M, int64_t N, int64_t K, const T* A, int64_t lda, int64_t seg, int64_t seg_stride,
          const T* B, int64_t ldb, T* C, int64_t ldc, bool accumulate) {
    if (M <= 0 || N <= 0) return;
    FPM_CHECK_ARG(t != nullptr, "no CPU team");
    FPM_CHECK_ARG(seg >= 1, "segment length must be >= 1");
    if (K <= 0) {
        if (!accumulate)
            for (int64_t i = 0; i < M; ++i) std::memset(C + i * ldc, 0, (size_t)N * sizeof(T));
        return;
    }
    const Kernel<T> kn = pick<T>();
    const int MR = kn.MR, NR = kn.NR;
    const int nt = t->n;
    const int64_t nc_max = std::min<int64_t>(NC, (N + NR - 1) / NR * NR);
    const size_t b_bytes = (size_t)KC * nc_max * sizeof(T);
    const int64_t mc = MC / MR * MR;
    const size_t a_bytes = (size_t)KC * mc * sizeof(T);
    if (t->b_cap < b_bytes) {
        std::free(t->b_buf);
        t->b_buf = aligned(b_bytes);
        t->b_cap = b_bytes;
    }
    for (int i = 0; i < nt; ++i)
        if (t->a_cap[i] < a_bytes) {
            std::free(t->a_buf[i]);
            t->a_buf[i] = aligned(a_bytes);
            t->a_cap[i] = a_bytes;
        }
    // rows per thread: whole MR panels, as even as possible ("x / c on each core")
    const int64_t panels = (M + MR - 1) / MR;
    auto A_at = [&](int64_t i, int64_t k) -> const T* {
        return A + (k / seg) * seg_stride + i * lda + (k % seg);
    };
    t->run([&](int tid, int n) {
        const int64_t p0 = panels * tid / n, p1 = panels * (tid + 1) / n;
        const int64_t r0 = std::min(M, p0 * MR), r1 = std::min(M, p1 * MR);
        T* bp = static_cast<T*>(t->b_buf);
        T* ap = static_cast<T*>(t->a_buf[tid]);
        alignas(64) T tile[12 * 32];
        for (int64_t jc = 0; jc < N; jc += NC) {
            const int64_t nc = std::min(NC, N - jc);
            const int64_t npan = (nc + NR - 1) / NR;
            for (int64_t pc = 0; pc < K; pc += KC) {
                const int64_t kc = std::min(KC, K - pc);
                // pack B(pc.., jc..) into NR-wide micro-panels [k][NR], zero-padded
                for (int64_t jp = npan * tid / n; jp < npan * (tid + 1) / n; ++jp) {
                    T* dst = bp + jp * NR * kc;
                    const int64_t j0 = jc + jp * NR, w = std::min<int64_t>(NR, N - j0);
                    for (int64_t k = 0; k < kc; ++k) {
                        const T* src = B + (pc + k) * ldb + j0;
                        T* d = dst + k * NR;
                        std::memcpy(d, src, (size_t)w * sizeof(T));
                        for (int64_t j = w; j < NR; ++j) d[j] = T(0);
                    }
                }
                t->barrier();
                const bool load_c = accumulate || pc > 0;
                for (int64_t ic = r0; ic < r1; ic += mc) {
                    const int64_t m = std::min(mc, r1 - ic);
                    const int64_t mpan = (m + MR - 1) / MR;
                    // pack A(ic.., pc..) into MR-tall micro-panels [k][MR], zero-padded
                    for (int64_t ip = 0; ip < mpan; ++ip) {
                        T* dst = ap + ip * MR * kc;
                        for (int i = 0; i < MR; ++i) {
                            const int64_t row = ic + ip * MR + i;
                            if (row >= ic + m) {
                                for (int64_t k = 0; k < kc; ++k) dst[k * MR + i] = T(0);
                                continue;
                            }
                            int64_t k = 0;
                            while (k < kc) {  // contiguous runs inside one K segment
                                const int64_t kk = pc + k;
                                const int64_t run = std::min<int64_t>(kc - k, seg - kk % seg);
                                const T* src = A_at(row, kk);
                                for (int64_t r = 0; r < run; ++r) dst[(k + r) * MR + i] = src[r];
                                k += run;
                            }
                        }
                    }
                    for (int64_t jp = 0; jp < npan; ++jp) {
                        const int64_t j0 = jc + jp * NR, w = std::min<int64_t>(NR, N - j0);
                        const T* bpan = bp + jp * NR * kc;
                        for (int64_t ip = 0; ip < mpan; ++ip) {
                            const int64_t i0 = ic + ip * MR, h = std::min<int64_t>(MR, ic + m - i0);
                            T* c = C + i0 * ldc + j0;
                            if (h == MR && w == NR) {
                                kn.uk(kc, ap + ip * MR * kc, bpan, c, ldc, load_c);
                            } else {  // edge tile: same sums into a scratch tile, then C = C + tile
                                kn.uk(kc, ap + ip * MR * kc, bpan, tile, NR, false);
                                for (int64_t i = 0; i < h; ++i)
                                    for (int64_t j = 0; j < w; ++j)
                                        c[i * ldc + j] = load_c ? c[i * ldc + j] + tile[i * NR + j] : tile[i * NR + j];
                            }
                        }
                    }
                }
                t->barrier();  // nobody still reads this B block
            }
        }
    });
}

}  // namespace

const char* isa() { return have_avx512() ? "avx512" : (have_avx2() ? "avx2" : "generic"); }

void gemm_f32(Team* t, int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, int64_t seg, int64_t seg_stride,
              const float* B, int64_t ldb, float* C, int64_t ldc, bool accumulate) {
    gemm<float>(t, M, N, K, A, lda, seg, seg_stride, B, ldb, C, ldc, accumulate);
}
void gemm_f64(Team* t, int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, int64_t seg, int64_t seg_stride,
              const double* B, int64_t ldb, double* C, int64_t ldc, bool accumulate) {
    gemm<double>(t, M, N, K, A, lda, seg, seg_stride, B, ldb, C, ldc, accumulate);
}

// ------------------------------------------------------------------ generator
namespace {
inline uint64_t synth_hash_host(uint64_t seed, uint64_t idx) {
    const uint64_t key = seed * 0xD1B54A32D192ED03ull;
    uint64_t z = key + (idx + 1) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
}  // namespace

void fill_synthetic(Team* t, void* dst, bool f64, int64_t ld, uint64_t seed, int64_t N, int64_t r0, int64_t c0,
                    int64_t rows, int64_t cols, int dist) {
    FPM_CHECK_ARG(dist == 0 || dist == 1, "unknown distribution %d", dist);
    auto body = [&](int tid, int n) {
        for (int64_t i = rows * tid / n; i < rows * (tid + 1) / n; ++i)
            for (int64_t j = 0; j < cols; ++j) {
                const uint64_t z = synth_hash_host(seed, (uint64_t)(r0 + i) * (uint64_t)N + (uint64_t)(c0 + j));
                const double x = dist == 0 ? (double)(z >> 40) * 0x1p-23 - 1.0 : (double)((z >> 32) % 17) - 8.0;
                if (f64) static_cast<double*>(dst)[i * ld + j] = x;
                else static_cast<float*>(dst)[i * ld + j] = (float)x;
            }
    };
    if (t) t->run(body);
    else body(0, 1);
}

}  // namespace cpu
}  // namespace fpm

// ===================================================================== C ABI
extern "C" int fpm_k_cpu_gemm(int32_t dt, int64_t M, int64_t N, int64_t K, const void* A, int64_t lda, int64_t seg,
                              int64_t seg_stride, const void* B, int64_t ldb, void* C, int64_t ldc,
                              int32_t accumulate, int32_t threads, int32_t pin) {
    return fpm::guarded([&] {
        FPM_CHECK_ARG(dt == FPM_F32 || dt == FPM_F64, "bad dtype");
        FPM_CHECK_ARG(M >= 0 && N >= 0 && K >= 0, "negative shape");
        FPM_CHECK_ARG(threads >= 1 && threads <= 1024, "threads must be in [1, 1024]");
        FPM_CHECK_ARG((M == 0 || N == 0) || (A && B && C), "null matrix");
        FPM_CHECK_ARG(lda >= 0 && ldb >= N && ldc >= N, "bad leading dimension");
        std::vector<int> cores;
        if (pin) {
            cores = fpm::cpu::allowed_cores();
            FPM_CHECK_ARG((int)cores.size() >= threads, "only %zu cores in the affinity mask", cores.size());
            cores.resize(threads);
        }
        std::unique_ptr<fpm::cpu::Team, void (*)(fpm::cpu::Team*)> team(fpm::cpu::team_create(cores, threads),
                                                                         fpm::cpu::team_destroy);
        if (seg <= 0) seg = std::max<int64_t>(K, 1);
        if (dt == FPM_F32)
            fpm::cpu::gemm_f32(team.get(), M, N, K, static_cast<const float*>(A), lda, seg, seg_stride,
                               static_cast<const float*>(B), ldb, static_cast<float*>(C), ldc, accumulate != 0);
        else
            fpm::cpu::gemm_f64(team.get(), M, N, K, static_cast<const double*>(A), lda, seg, seg_stride,
                               static_cast<const double*>(B), ldb, static_cast<double*>(C), ldc, accumulate != 0);
    });
}

extern "C" int fpm_cpu_isa(char* out, int32_t cap) {
    return fpm::guarded([&] {
        FPM_CHECK_ARG(out != nullptr && cap >= 1, "null buffer");
        std::snprintf(out, (size_t)cap, "%s", fpm::cpu::isa());
    });
}

extern "C" int fpm_cpu_cores(int32_t* cores_out, int32_t cap, int32_t* count) {
    return fpm::guarded([&] {
        FPM_CHECK_ARG(count != nullptr && (cap == 0 || cores_out != nullptr), "null argument");
        const std::vector<int> c = fpm::cpu::allowed_cores();
        for (int i = 0; i < (int)c.size() && i < cap; ++i) cores_out[i] = c[i];
        *count = (int32_t)c.size();
    });
}
