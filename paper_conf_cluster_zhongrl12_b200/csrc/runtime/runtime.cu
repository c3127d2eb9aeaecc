// Runtime of the FPM-partitioned column-based parallel matrix multiplication
// (§IV): device contexts, resident data layout, the N/b
// iteration loop with look-ahead pivot exchange, kernel-based speed sampling
// (fpm_sample) and the C ABI of the runtime part.
//
// Per device and iteration k (slot = k mod 2, look-ahead one iteration):
//   comm stream:    wait free[slot] -> receive A(rows_i, k), B(k, cols_i)
//                   (local copies or NCCL) -> split / transpose into the slot's
//                   operand buffers -> record ready[slot]
//   compute stream: wait ready[slot] -> rank-b update C_i += A(b) B(b) ->
//                   record free[slot]
// so the exchange and staging of k+1 run under the update of k (P:40/P:68
// overlap principle; "broadcast horizontally and vertically").
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <exception>
#include <condition_variable>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

#include "../common.hpp"
#include "../host/cpu_device.hpp"
#include "../host/host_algos.hpp"
#include "../kernels/kernels.hpp"
#include "green.hpp"
#include "nccl_loader.hpp"

#define CU(expr)                                                                                        \
    do {                                                                                                \
        cudaError_t _e = (expr);                                                                        \
        if (_e != cudaSuccess)                                                                          \
            ::fpm::fail(FPM_ECUDA, "%s: %s (%s:%d)", #expr, cudaGetErrorString(_e), __FILE__, __LINE__); \
    } while (0)
#define NC(expr)                                                                                   \
    do {                                                                                           \
        ncclResult_t _r = (expr);                                                                  \
        if (_r != ncclSuccess)                                                                     \
            ::fpm::fail(FPM_ENCCL, "%s: %s", #expr, ::fpm::nccl().GetErrorString(_r));             \
    } while (0)

namespace fpm {

// Out-of-core C (GPU kernel versions 2/3): when C_i
// exceeds the device's memory budget for it, C_i lives in pinned host memory and
// every update streams it through the device in row bands held in a ring of R
// device buffers (R = 2 is the paper's "C0 and C1"): the H2D of a later
// band and the D2H of an earlier one overlap the update of the current band on
// three streams.
constexpr int kMaxBandBufs = 16;
constexpr int kMaxTail = 16;             // groups of the download-overlapped tail
constexpr int kSlots = 3 + kMaxTail;     // operand slots per device
constexpr int kFusedSlot = kSlots - 1;  // the fused tail: all tail pivots as one operand
struct Ring {
    int R;         // buffers in use
    int64_t rows;  // rows per band
};
struct BandPipe {
    cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
    cudaEvent_t in[kMaxBandBufs] = {}, done[kMaxBandBufs] = {}, out[kMaxBandBufs] = {};
    void* buf[kMaxBandBufs] = {};
    bool used[kMaxBandBufs] = {};
    int nbuf = 0;                         // R
    size_t buf_bytes = 0;
    int next = 0, dir = 1;                // ring position and direction (reverses with the band order)
    int last = -1;                        // buffer of the most recent device -> host copy
    int last_step = -1;                   // buffer used by the most recent update
    std::vector<cudaEvent_t> out_band;    // D2H of band j done (its host rows are current)
    std::vector<char> band_used;
    int64_t bytes = 0;                    // host <-> device bytes issued
};

struct Device {
    int idx = 0;       // index in the arrangement (= rank in NCCL mode)
    int cuda_dev = 0;
    int sm_cap = 0;    // 0 = all SMs
    int num_sms = 0;   // persistent grid of the update kernel
    GreenPartition green;  // SM partition (option "sm_partition" = 1), else none
    int64_t c_cap = 0;     // bytes of device memory C_i may use (0 = no limit)
    bool ooc = false;      // C_i out of core for the current problem
    float* hC = nullptr;   // pinned host C_i (H x W) when out of core
    std::vector<void*> host_allocs;
    BandPipe bp;
    Ring ring{0, 0};       // out-of-core band geometry of the current problem
    int64_t g_ooc_bytes = 0;        // out-of-core bytes of one captured k-loop
    cudaEvent_t ev_join[4] = {};    // graph capture: join of this device's streams
    cudaStream_t s_comp = nullptr, s_comm = nullptr;
    cudaStream_t s_up = nullptr;  // pmm_run: host -> device panel uploads, run ahead of the staging
    cudaEvent_t ev_ready[kSlots] = {}, ev_free[kSlots] = {};
    cudaEvent_t ev_start = nullptr, ev_stop = nullptr, ev_io0 = nullptr, ev_io1 = nullptr;
    std::vector<cudaEvent_t> ev_pack0, ev_pack1, ev_upd0, ev_upd1, ev_up;

    // problem state
    colpart_rect rect{-1, 0, 0, 0, 0};
    int64_t H = 0, W = 0;  // rectangle in elements
    void* A = nullptr;     // w block-columns, each H x b row-major (K-major panels)
    void* B = nullptr;     // H x W row-major (h block-rows of b x W)
    // IPC: upload progress of this rank's panels, at the end of B's allocation
    // (so peers map it with B): (epoch << 16) | (k + 1) once panels 0..k landed
    uint64_t* up_flag = nullptr;
    void* C = nullptr;     // H x W row-major
    // operand slots: 0, 1 double-buffer the k-loop; 2 .. 2+tail_slots-1 hold the
    // groups of the download-overlapped tail (compute_into, allocated on demand)
    void* a_recv[kSlots] = {}, *b_recv[kSlots] = {};
    void* bt[kSlots] = {};                  // W x b (K-major) transposed B pivot row
    void* a_hi[kSlots] = {}, *a_lo[kSlots] = {}, *b_hi[kSlots] = {}, *b_lo[kSlots] = {};
    float* sa[kSlots] = {}, *sb[kSlots] = {};
    const void* a_op[kSlots] = {};          // FP64: A operand of the slot
    int b_from[kSlots] = {};                // FP32 slots 0, 1: device whose staged B operand this slot's
                                            // update reads (its own index, or the column's B owner on the
                                            // same GPU: option "share_b")
    int tail_slots = 0;                     // slots 2.. allocated
    // fused tail (kFusedSlot): the tail's pivots staged as one K = tail_K operand
    // with common F16X3 scales (maxima merged in tmax_a / tmax_b first)
    int64_t tail_K = 0, tail_K_alloc = 0;
    unsigned* tmax_a = nullptr;
    unsigned* tmax_b = nullptr;
    std::vector<void*> tail_allocs;
    cudaEvent_t ev_tpack0 = nullptr, ev_tpack1 = nullptr;  // staging of the fused tail (second pass)
    bool tail_fused_run = false;  // the current k-loop stages its tail into kFusedSlot
    // in-kernel staging (option "fused_staging"): update g stages group g + 1
    // with its staging warp; B column maxima and the grid-barrier counters
    bool fs_run = false;
    unsigned* stg_bmax = nullptr;
    unsigned* stg_ctr = nullptr;
    // band-streamed tail (pmm_run, one device holding all of A and B): the tail's
    // A rows arrive band by band into tail_rows (H x tail_K, row-major)
    bool tail_streamed_run = false;
    float* tail_rows = nullptr;
    std::vector<cudaEvent_t> ev_band_up, ev_band_st;  // per band: rows uploaded, rows staged
    cudaEvent_t ev_tail_b = nullptr;                  // tail B rows uploaded
    std::vector<void*> allocs;
    int64_t launches = 0;                   // library kernels launched (running count)

    // host-CPU device (cuda_dev = FPM_CPU_DEVICE; a socket
    // of c cores running the GEMM kernel together): A_i, B_i, C_i in host memory
    // (pinned and mapped when the context has GPUs, so their staging kernels read
    // this device's pivots directly), its update on a team of pinned cores
    bool cpu = false;
    int cores = 0;                          // c
    int first_core = -1;                    // index of its first core in the affinity mask
    cpu::Team* team = nullptr;
    std::vector<void*> plain_allocs;        // host memory without a GPU in the context
    void* h_arecv[2] = {}, *h_brecv[2] = {}; // gathered pivots of a group
    std::vector<std::pair<int, cudaStream_t>> pulls;  // (CUDA ordinal, stream) of device -> host pivot pulls
    std::vector<double> cpu_pack_s, cpu_upd_s;         // per group, last k-loop
    double cpu_loop_s = 0.0;                // last k-loop, wall time
    int64_t cpu_bytes = 0;                  // pivot bytes received in the last k-loop

    bool live() const { return H > 0 && W > 0; }
};

}  // namespace fpm

struct pmm_ctx {
    bool nccl_mode = false;  // one process per GPU, pivots over NCCL
    bool ipc_mode = false;   // one process per GPU, pivots pulled from peers' memory (CUDA IPC)
    int rank = 0, world = 1;
    std::vector<fpm::Device> devs;
    ncclComm_t world_comm = nullptr;
    ncclComm_t col_comm = nullptr;
    std::vector<int> col_members;  // global ranks of my column, sorted
    // IPC mode: peers' resident A_q, B_q mapped into this process
    std::vector<void*> peer_A, peer_B;
    std::vector<uint64_t*> peer_flag;  // peers' upload-progress flags (streamed pmm_run)
    bool peers_ready = false;
    uint64_t epoch = 0;                // streamed runs issued (the same sequence on every rank)

    bool have_problem = false;
    int64_t N = 0, b = 0, n = 0;
    int p = 0;
    fpm_dtype dt = FPM_F32;
    std::vector<colpart_rect> rects;
    std::vector<std::vector<fpm::Move>> plan_a, plan_b;

    int f32_scheme = -1;  // fpm::SplitScheme, -1 = auto (scheme_for)
    int cta_group = 2;
    int raster_group = 0;  // 0 = auto: 16 (F16I8 12, measured c5) x the device's share of its GPU's SMs
    int l2_hint_b = 0;
    int kernel_variant = -1;  // auto
    int chunk_k = 0;          // F16X3 / TF32X3 default kernel: K per TMEM accumulation (0 auto = 512)
    int raster_snake = 0;     // F16X3 / TF32X3 default kernel: serpentine raster over groups
    double sample_rel_ci = 0.025;  // fpm_sample stop rule: 95 % half-width / mean (Q8)
    int share_b = 1;          // local FP32: column members on the B owner's GPU read its staged B operand
    int fuse = 0;             // pivots per update (0 = auto)
    int fuse_max = 1;         // resolved for the current problem
    int ooc_keep = 1;         // out-of-core: keep the last R bands, reverse every other update
    int graph = 1;            // pmm_compute replays the k-loop as one CUDA graph
    cudaGraphExec_t gexec = nullptr;
    cudaEvent_t ev_fork = nullptr;  // on devs[0]'s device
    int64_t g_bytes = 0, g_launches = 0;
    int e2e_tail = -1;        // groups of the download-overlapped tail (-1 auto, 0 off)
    int64_t tail_band = 2048; // rows of C_i per band of the tail (multiple of 256)
    int tail_fuse = 1;        // local / IPC FP32: the tail as one fused operand (1) or per group (0)
    int fused_staging = 1;    // FP32 F16X3 k-loop: the update kernel stages the next group
    bool stream_flags = false;  // this streamed run writes upload-progress flags (in-kernel staging)
    int tail_stream = 1;      // pmm_run on one device: the tail's B rows first, its A rows band by band
    int sm_partition = 0;     // 0: SM caps as persistent grid sizes; 1: green-context partitions
    int ooc_buffers = 8;      // out-of-core: up to R band buffers in the C cap (2 = the paper's C0, C1)
    std::vector<std::pair<int64_t, int>> groups;  // (first pivot, pivots) of each update
    std::vector<std::pair<int64_t, int>> groups_streamed;  // the same for pmm_run (host-streamed inputs)
};

namespace fpm {
namespace {

size_t esize(fpm_dtype dt) { return dt == FPM_F64 ? 8 : 4; }

void* dalloc(Device& d, size_t bytes) {
    if (bytes == 0) return nullptr;
    void* p = nullptr;
    cudaError_t e = cudaMalloc(&p, bytes);
    if (e != cudaSuccess) {
        cudaGetLastError();
        fail(FPM_ENOMEM, "cudaMalloc(%zu) on device %d: %s", bytes, d.cuda_dev, cudaGetErrorString(e));
    }
    d.allocs.push_back(p);
    return p;
}

void* halloc(Device& d, size_t bytes, unsigned flags = cudaHostAllocPortable) {
    void* p = nullptr;
    cudaError_t e = cudaHostAlloc(&p, bytes, flags);
    if (e != cudaSuccess) {
        cudaGetLastError();
        fail(FPM_ENOMEM, "cudaHostAlloc(%zu): %s", bytes, cudaGetErrorString(e));
    }
    d.host_allocs.push_back(p);
    return p;
}

// Memory of a CPU device: pinned and mapped (device-accessible through its UVA
// address, so GPU devices' staging kernels pull its pivots directly) when the
// context drives GPUs, plain aligned host memory otherwise.
void* cpu_mem(Device& d, size_t bytes, bool pinned) {
    if (bytes == 0) return nullptr;
    if (pinned) return halloc(d, bytes, cudaHostAllocPortable | cudaHostAllocMapped);
    void* p = nullptr;
    if (posix_memalign(&p, 64, bytes) != 0) fail(FPM_ENOMEM, "host allocation of %zu bytes failed", bytes);
    d.plain_allocs.push_back(p);
    return p;
}

void bp_init(BandPipe& bp) {
    CU(cudaStreamCreateWithFlags(&bp.s_h2d, cudaStreamNonBlocking));
    CU(cudaStreamCreateWithFlags(&bp.s_d2h, cudaStreamNonBlocking));
    for (int i = 0; i < kMaxBandBufs; ++i)
        for (cudaEvent_t* e : {&bp.in[i], &bp.done[i], &bp.out[i]})
            CU(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
}

void bp_release_bands(BandPipe& bp) {
    for (cudaEvent_t e : bp.out_band) cudaEventDestroy(e);
    bp.out_band.clear();
    bp.band_used.clear();
    for (int i = 0; i < kMaxBandBufs; ++i) {
        bp.buf[i] = nullptr;
        bp.used[i] = false;
    }
    bp.nbuf = 0;
    bp.buf_bytes = 0;
    bp.next = 0;
    bp.dir = 1;
    bp.last = bp.last_step = -1;
}

void bp_destroy(BandPipe& bp) {
    bp_release_bands(bp);
    for (int i = 0; i < kMaxBandBufs; ++i)
        for (cudaEvent_t e : {bp.in[i], bp.done[i], bp.out[i]})
            if (e) cudaEventDestroy(e);
    if (bp.s_h2d) cudaStreamDestroy(bp.s_h2d);
    if (bp.s_d2h) cudaStreamDestroy(bp.s_d2h);
    bp = BandPipe{};
}

// Ring geometry for an H x W C (element size es) in `cap` bytes with up to R
// buffers: bands of whole multiples of 256 rows (one CTA-pair tile row), at
// least 256; fewer buffers (not below 2) when R bands of 256 rows would not fit.
Ring ring_for(int64_t cap, int64_t H, int64_t W, size_t es, int R) {
    const int64_t row_bytes = W * (int64_t)es;
    const int r = (int)std::min<int64_t>(R, std::max<int64_t>(2, cap / (256 * row_bytes)));
    const int64_t rows = std::max<int64_t>(256, cap / r / row_bytes / 256 * 256);
    return {r, std::min(rows, H)};
}

// Allocate the R band buffers (bytes each) and the per-band events.
void bp_alloc_bands(Device& owner, BandPipe& bp, int R, size_t bytes, int64_t nbands) {
    bp_release_bands(bp);
    FPM_CHECK_ARG(R >= 2 && R <= kMaxBandBufs, "out-of-core buffers must be in [2, %d]", kMaxBandBufs);
    for (int i = 0; i < R; ++i) bp.buf[i] = dalloc(owner, bytes);
    bp.nbuf = R;
    bp.buf_bytes = bytes;
    bp.out_band.resize(nbands);
    for (auto& e : bp.out_band) CU(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    bp.band_used.assign(nbands, 0);
}

// One out-of-core update of the host matrix hC (H rows of row_bytes, packed):
// for each band of `band_rows` rows, H2D (only if `accumulate`) on s_h2d,
// update on s_comp via launch(r0, rows, device band), D2H on s_d2h.  A band's
// H2D waits for the D2H of the buffer's previous occupant (reuse) and for the
// previous D2H of the same band (its host rows).
//
// P:34 "we keep the last two rectangles accumulating intermediate results in
// the device in each iteration and reverse the updating order every other
// iteration, which can save two transfers in each direction", generalised to
// R buffers (the paper's R = 2): `reverse` runs the bands last to first;
// `keep_tail` leaves the last min(R, bands) bands of this call in their buffers
// (no D2H); `kept_head` says the previous call kept its tail, so this call (in
// the opposite order) starts on those bands without H2D.  The ring then runs
// backwards: the buffer freed first (its band updated and copied out first) is
// the one the first non-resident band needs.  Returns the launches issued.
struct BandCall {
    bool accumulate = true;
    bool reverse = false;
    bool kept_head = false;
    bool keep_tail = false;
};

template <class Launch>
int64_t banded_update(BandPipe& bp, const Ring& ring, char* hC, int64_t H, size_t row_bytes, const BandCall& bc,
                      cudaStream_t s_comp, Launch&& launch) {
    const int R = ring.R;
    const int64_t band_rows = ring.rows;
    const int64_t nb = (H + band_rows - 1) / band_rows;
    if (R < 2 || R > bp.nbuf || (int64_t)bp.out_band.size() < nb || (size_t)band_rows * row_bytes > bp.buf_bytes)
        fail(FPM_ESTATE, "band pipeline not sized for %lld bands of %lld rows", (long long)nb,
             (long long)band_rows);
    if (bp.next >= R) bp.next = 0;
    const int64_t nkeep = std::min<int64_t>(R, nb);
    if (bc.kept_head) {  // start on the previous call's last band, walk the ring the other way
        bp.dir = -bp.dir;
        bp.next = bp.last_step;
    }
    int64_t launches = 0;
    for (int64_t t = 0; t < nb; ++t) {
        const int64_t j = bc.reverse ? nb - 1 - t : t;
        const int buf = bp.next;
        bp.next = ((bp.next + bp.dir) % R + R) % R;
        const int64_t r0 = j * band_rows, rows = std::min(band_rows, H - r0);
        const size_t bytes = (size_t)rows * row_bytes;
        const bool resident = bc.kept_head && t < nkeep;  // already in `buf`, current
        if (!resident) {
            if (bp.used[buf]) {  // previous occupant updated and (unless kept) copied out
                CU(cudaStreamWaitEvent(bp.s_h2d, bp.done[buf], 0));
                CU(cudaStreamWaitEvent(bp.s_h2d, bp.out[buf], 0));
            }
            if (bc.accumulate) {
                if (bp.band_used[j]) CU(cudaStreamWaitEvent(bp.s_h2d, bp.out_band[j], 0));
                CU(cudaMemcpyAsync(bp.buf[buf], hC + (size_t)r0 * row_bytes, bytes, cudaMemcpyHostToDevice,
                                   bp.s_h2d));
                bp.bytes += (int64_t)bytes;
            }
            CU(cudaEventRecord(bp.in[buf], bp.s_h2d));
            CU(cudaStreamWaitEvent(s_comp, bp.in[buf], 0));
        }
        launch(r0, rows, bp.buf[buf]);
        ++launches;
        bp.used[buf] = true;
        bp.last_step = buf;
        CU(cudaEventRecord(bp.done[buf], s_comp));
        if (bc.keep_tail && t >= nb - nkeep) continue;  // stays in the buffer for the next call
        CU(cudaStreamWaitEvent(bp.s_d2h, bp.done[buf], 0));
        CU(cudaMemcpyAsync(hC + (size_t)r0 * row_bytes, bp.buf[buf], bytes, cudaMemcpyDeviceToHost, bp.s_d2h));
        bp.bytes += (int64_t)bytes;
        CU(cudaEventRecord(bp.out[buf], bp.s_d2h));
        CU(cudaEventRecord(bp.out_band[j], bp.s_d2h));
        bp.band_used[j] = 1;
        bp.last = buf;
    }
    return launches;
}

// Make `s` wait until every host copy of the band pipeline has landed.
void bp_join(BandPipe& bp, cudaStream_t s) {
    if (bp.last >= 0) CU(cudaStreamWaitEvent(s, bp.out[bp.last], 0));
}

void free_problem(Device& d) {
    if (d.cpu) {
        for (auto& ps : d.pulls) cudaStreamSynchronize(ps.second);
        for (void* p : d.plain_allocs) std::free(p);
        d.plain_allocs.clear();
        for (void* p : d.host_allocs) cudaFreeHost(p);
        d.host_allocs.clear();
        d.A = d.B = d.C = nullptr;
        for (int s = 0; s < 2; ++s) d.h_arecv[s] = d.h_brecv[s] = nullptr;
        d.H = d.W = 0;
        return;
    }
    cudaSetDevice(d.cuda_dev);
    if (d.bp.s_d2h) cudaStreamSynchronize(d.bp.s_d2h);
    bp_release_bands(d.bp);
    for (void* p : d.allocs) cudaFree(p);
    d.allocs.clear();
    for (void* p : d.host_allocs) cudaFreeHost(p);
    d.host_allocs.clear();
    d.hC = nullptr;
    d.ooc = false;
    for (auto* v : {&d.ev_pack0, &d.ev_pack1, &d.ev_upd0, &d.ev_upd1, &d.ev_up}) {
        for (cudaEvent_t e : *v) cudaEventDestroy(e);
        v->clear();
    }
    d.A = d.B = d.C = nullptr;
    d.up_flag = nullptr;
    d.tail_slots = 0;
    for (void* p : d.tail_allocs) cudaFree(p);
    d.tail_allocs.clear();
    d.tail_K = d.tail_K_alloc = 0;
    d.tmax_a = d.tmax_b = nullptr;
    d.tail_rows = nullptr;
    d.stg_bmax = d.stg_ctr = nullptr;
    d.fs_run = false;
    for (int s = 0; s < kSlots; ++s) {
        d.a_recv[s] = d.b_recv[s] = d.bt[s] = d.a_hi[s] = d.a_lo[s] = d.b_hi[s] = d.b_lo[s] = nullptr;
        d.sa[s] = d.sb[s] = nullptr;
        d.a_op[s] = nullptr;
    }
    d.H = d.W = 0;
}

void init_device(Device& d) {
    if (d.cpu) {  // a team of c worker threads pinned to its cores (P:10 (i))
        const std::vector<int> all = cpu::allowed_cores();
        if (d.cores < 1 || d.first_core < 0 || d.first_core + d.cores > (int)all.size())
            fail(FPM_EUNSUPPORTED, "CPU device %d: cores [%d, %d) outside the %zu cores of the affinity mask", d.idx,
                 d.first_core, d.first_core + d.cores, all.size());
        d.team = cpu::team_create(std::vector<int>(all.begin() + d.first_core, all.begin() + d.first_core + d.cores));
        return;
    }
    CU(cudaSetDevice(d.cuda_dev));
    int sms = 0;
    CU(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, d.cuda_dev));
    if (d.sm_cap != 0) {
        if (d.sm_cap < 2 || d.sm_cap % 2 != 0 || d.sm_cap > sms)
            fail(FPM_EUNSUPPORTED, "SM cap %d not achievable (even, in [2, %d]: CTA pairs)", d.sm_cap, sms);
        d.num_sms = d.sm_cap;
    } else {
        d.num_sms = sms;
    }
    if (d.green.ctx) {  // every kernel of this device (update, staging, NCCL) inside its SMs
        d.num_sms = d.green.sms;
        d.s_comp = green_stream(d.green);
        d.s_comm = green_stream(d.green);
    } else {
        CU(cudaStreamCreateWithFlags(&d.s_comp, cudaStreamNonBlocking));
        CU(cudaStreamCreateWithFlags(&d.s_comm, cudaStreamNonBlocking));
    }
    CU(cudaStreamCreateWithFlags(&d.s_up, cudaStreamNonBlocking));  // copies only: no SM partition
    for (int s = 0; s < kSlots; ++s) {
        CU(cudaEventCreateWithFlags(&d.ev_ready[s], cudaEventDisableTiming));
        CU(cudaEventCreateWithFlags(&d.ev_free[s], cudaEventDisableTiming));
    }
    CU(cudaEventCreate(&d.ev_start));
    CU(cudaEventCreate(&d.ev_stop));
    CU(cudaEventCreate(&d.ev_io0));
    CU(cudaEventCreate(&d.ev_io1));
    CU(cudaEventCreate(&d.ev_tpack0));
    CU(cudaEventCreate(&d.ev_tpack1));
    for (auto& e : d.ev_join) CU(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    bp_init(d.bp);
}

void destroy_device(Device& d) {
    free_problem(d);
    if (d.cpu) {
        for (auto& ps : d.pulls) {
            cudaSetDevice(ps.first);
            cudaStreamDestroy(ps.second);
        }
        d.pulls.clear();
        cpu::team_destroy(d.team);
        d.team = nullptr;
        return;
    }
    cudaSetDevice(d.cuda_dev);
    bp_destroy(d.bp);
    for (int s = 0; s < kSlots; ++s) {
        if (d.ev_ready[s]) cudaEventDestroy(d.ev_ready[s]);
        if (d.ev_free[s]) cudaEventDestroy(d.ev_free[s]);
    }
    for (cudaEvent_t e : {d.ev_start, d.ev_stop, d.ev_io0, d.ev_io1, d.ev_tpack0, d.ev_tpack1, d.ev_tail_b})
        if (e) cudaEventDestroy(e);
    for (auto* v : {&d.ev_band_up, &d.ev_band_st}) {
        for (cudaEvent_t e : *v) cudaEventDestroy(e);
        v->clear();
    }
    d.ev_tail_b = nullptr;
    for (auto& e : d.ev_join) {
        if (e) cudaEventDestroy(e);
        e = nullptr;
    }
    if (d.s_comp) cudaStreamDestroy(d.s_comp);
    if (d.s_comm) cudaStreamDestroy(d.s_comm);
    if (d.s_up) cudaStreamDestroy(d.s_up);
    d.s_comp = d.s_comm = d.s_up = nullptr;
    for (int s = 0; s < kSlots; ++s) d.ev_ready[s] = d.ev_free[s] = nullptr;
    d.ev_start = d.ev_stop = d.ev_io0 = d.ev_io1 = d.ev_tpack0 = d.ev_tpack1 = nullptr;
    green_destroy(d.green);
}


// Timing events: while the k-loop is being captured into a CUDA graph they must
// become event-record nodes (cudaEventRecordExternal), not capture-internal
// dependencies, so that replays still time each group.
bool g_capturing = false;
void rec_t(cudaEvent_t e, cudaStream_t s) {
    CU(cudaEventRecordWithFlags(e, s, g_capturing ? cudaEventRecordExternal : cudaEventRecordDefault));
}

float elapsed_ms(cudaEvent_t a, cudaEvent_t b) {
    float ms = 0.0f;
    CU(cudaEventElapsedTime(&ms, a, b));
    return ms;
}

Device* local_dev(pmm_ctx* ctx, int idx) {
    for (auto& d : ctx->devs)
        if (d.idx == idx) return &d;
    return nullptr;
}

// ------------------------------------------------------------------ IPC peers
void close_peers(pmm_ctx* ctx) {
    if (!ctx->ipc_mode) return;
    if (!ctx->devs.empty()) cudaSetDevice(ctx->devs[0].cuda_dev);
    for (auto* v : {&ctx->peer_A, &ctx->peer_B})
        for (void*& ptr : *v) {
            if (ptr) cudaIpcCloseMemHandle(ptr);
            ptr = nullptr;
        }
    std::fill(ctx->peer_flag.begin(), ctx->peer_flag.end(), nullptr);
    ctx->peers_ready = false;
}

// The captured k-loop refers to the problem's buffers, events and options.
void drop_graph(pmm_ctx* ctx) {
    if (ctx->gexec) cudaGraphExecDestroy(ctx->gexec);
    ctx->gexec = nullptr;
}

// Option "sm_partition": rebuild every device's streams, inside disjoint
// green-context SM partitions of its cap (on) or on the whole GPU (off).
void set_sm_partition(pmm_ctx* ctx, bool green) {
    drop_graph(ctx);
    // carve the partitions first: a failure leaves the context as it was
    std::vector<GreenPartition> parts(ctx->devs.size());
    if (green) {
        for (auto& d : ctx->devs)
            if (!d.cpu && d.sm_cap == 0)
                fail(FPM_EUNSUPPORTED, "sm_partition = 1 needs an SM cap on every device (device %d has none)", d.idx);
        try {
            std::vector<int> gpus;
            for (auto& d : ctx->devs)
                if (!d.cpu && std::find(gpus.begin(), gpus.end(), d.cuda_dev) == gpus.end()) gpus.push_back(d.cuda_dev);
            for (int g : gpus) {  // one split per GPU: the partitions of its devices are disjoint
                std::vector<size_t> on;
                std::vector<int> caps;
                for (size_t i = 0; i < ctx->devs.size(); ++i)
                    if (!ctx->devs[i].cpu && ctx->devs[i].cuda_dev == g) {
                        on.push_back(i);
                        caps.push_back(ctx->devs[i].sm_cap);
                    }
                std::vector<GreenPartition> got = green_partitions(g, caps);
                for (size_t i = 0; i < on.size(); ++i) parts[on[i]] = got[i];
            }
        } catch (...) {
            for (auto& gp : parts) green_destroy(gp);
            throw;
        }
    }
    close_peers(ctx);
    for (auto& d : ctx->devs)
        if (!d.cpu) destroy_device(d);
        else free_problem(d);
    ctx->have_problem = false;
    for (size_t i = 0; i < ctx->devs.size(); ++i) {
        if (ctx->devs[i].cpu) continue;
        ctx->devs[i].green = parts[i];
        init_device(ctx->devs[i]);
    }
}

// Resident A_q / B_q of device q: local devices directly, IPC peers through the
// mapped handles.  These buffers are written only by upload/fill, never during
// the k-loop, so a pull needs no synchronisation with the owner.
const void* src_A(pmm_ctx* ctx, int q) {
    if (ctx->ipc_mode) return q == ctx->rank ? ctx->devs[0].A : ctx->peer_A[q];
    return local_dev(ctx, q)->A;
}
const void* src_B(pmm_ctx* ctx, int q) {
    if (ctx->ipc_mode) return q == ctx->rank ? ctx->devs[0].B : ctx->peer_B[q];
    return local_dev(ctx, q)->B;
}

// Stream memory operations (driver API, resolved at run time): the streamed
// IPC pmm_run orders a peer's pulls after this rank's uploads through a 64-bit
// progress flag in device memory instead of IPC events.
struct StreamMemOps {
    CUresult (*write64)(CUstream, CUdeviceptr, cuuint64_t, unsigned) = nullptr;
    CUresult (*wait64)(CUstream, CUdeviceptr, cuuint64_t, unsigned) = nullptr;
};
const StreamMemOps& stream_mem_ops() {
    static StreamMemOps ops;
    static bool done = false;
    if (!done) {
        cudaDriverEntryPointQueryResult q;
        void* p = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue64", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            ops.write64 = reinterpret_cast<decltype(ops.write64)>(p);
        p = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue64", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            ops.wait64 = reinterpret_cast<decltype(ops.wait64)>(p);
        cudaGetLastError();
        done = true;
    }
    if (!ops.write64 || !ops.wait64) fail(FPM_EUNSUPPORTED, "cuStreamWriteValue64 / cuStreamWaitValue64 unavailable");
    return ops;
}
uint64_t flag_value(uint64_t epoch, int64_t k) { return (epoch << 16) | (uint64_t)(k + 1); }

bool has_gpu(const pmm_ctx* ctx) {
    for (auto& d : ctx->devs)
        if (!d.cpu) return true;
    return false;
}
bool has_cpu(const pmm_ctx* ctx) {
    for (auto& d : ctx->devs)
        if (d.cpu) return true;
    return false;
}

// NCCL communicator configuration: the exchange runs beside the persistent
// update kernel, which holds every SM, so NCCL gets few CTAs (maxCTAs, env
// FPM_NCCL_MAX_CTAS, default 8) -- its transfers are NVLink-bound, not SM-bound.
ncclConfig_t nccl_config() {
    ncclConfig_t cfg = NCCL_CONFIG_INITIALIZER;
    int max_ctas = 8;
    if (const char* e = std::getenv("FPM_NCCL_MAX_CTAS")) max_ctas = std::max(1, std::atoi(e));
    cfg.minCTAs = 1;
    cfg.maxCTAs = max_ctas;
    return cfg;
}

// Wait for `ev` while polling the communicators for asynchronous errors (a peer
// that died or a network failure would otherwise block forever on the event).
void nccl_wait(pmm_ctx* ctx, cudaEvent_t ev) {
    const NcclApi& nc = nccl();
    for (int spin = 0;; ++spin) {
        const cudaError_t q = cudaEventQuery(ev);
        if (q == cudaSuccess) return;
        if (q != cudaErrorNotReady) CU(q);
        for (ncclComm_t c : {ctx->world_comm, ctx->col_comm}) {
            if (!c) continue;
            ncclResult_t ae = ncclSuccess;
            NC(nc.CommGetAsyncError(c, &ae));
            if (ae != ncclSuccess && ae != ncclInProgress) {
                nc.CommAbort(c);
                if (c == ctx->world_comm) ctx->world_comm = nullptr;
                else ctx->col_comm = nullptr;
                fail(FPM_ENCCL, "NCCL asynchronous error: %s (communicator aborted)", nc.GetErrorString(ae));
            }
        }
        if (spin > 64) std::this_thread::sleep_for(std::chrono::microseconds(200));
    }
}
// IPC contexts: wait for `ev` with a deadline.  The k-loop waits on peers'
// progress flags (stream waits, and the staging warps' acquire loads, which
// trap after 60 s); a peer process that stopped would otherwise block this
// rank forever.  Deadline: env FPM_IPC_TIMEOUT_S (default 600 s; 0 = none).
void ipc_wait(cudaEvent_t ev) {
    static const double limit = [] {
        const char* e = std::getenv("FPM_IPC_TIMEOUT_S");
        return e ? std::max(0.0, std::atof(e)) : 600.0;
    }();
    const auto t0 = std::chrono::steady_clock::now();
    for (int spin = 0;; ++spin) {
        const cudaError_t q = cudaEventQuery(ev);
        if (q == cudaSuccess) return;
        if (q != cudaErrorNotReady) CU(q);
        if (limit > 0 && std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() > limit)
            fail(FPM_ECUDA, "IPC k-loop unfinished after %.0f s: a peer's progress flag stopped advancing "
                            "(peer process stopped?); FPM_IPC_TIMEOUT_S sets the limit", limit);
        if (spin > 64) std::this_thread::sleep_for(std::chrono::microseconds(200));
    }
}

// A CPU device's stream for pulling pivots out of GPU `cuda_dev`'s memory.
cudaStream_t pull_stream(Device& d, int cuda_dev) {
    for (auto& ps : d.pulls)
        if (ps.first == cuda_dev) return ps.second;
    cudaStream_t s = nullptr;
    CU(cudaSetDevice(cuda_dev));
    CU(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    d.pulls.push_back({cuda_dev, s});
    return s;
}

// Raster group (tile-rows whose A panel stays in L2 while the B^T panel streams
// by) of device d's update: the option, else 16 (F16I8: 12) scaled by the
// device's share of the SMs of its GPU among this context's devices on it --
// devices that share a GPU share its L2, and their A groups must fit it together.
// Measured, c4 analogue (8 devices on one GPU, green partitions): group 16 on
// every device 65.6-67.6 % of the capped-aggregate peak, 8: 70.0, 4: 73.1, 2: 72.4.
int raster_group_for(const pmm_ctx* ctx, const Device& d, SplitScheme sch) {
    if (ctx->raster_group > 0) return ctx->raster_group;
    const int full = sch == SplitScheme::F16I8 ? 12 : 16;
    int sms_on_gpu = 0;
    for (const auto& q : ctx->devs)
        if (!q.cpu && q.cuda_dev == d.cuda_dev) sms_on_gpu += q.num_sms;
    if (sms_on_gpu <= d.num_sms) return full;
    return std::max(1, (int)std::lround((double)full * d.num_sms / sms_on_gpu));
}

// Pivots fused per update (FP32 only): option "fuse", 0 = auto = K of about 2048
// (measured on B200: f = 2 at b = 1024 gives 419 vs 392 TFLOP/s unfused and
// beats f = 3, 4; at b = 512, f = 2..8 give 404-406 vs 332 unfused).
int fuse_factor(pmm_ctx* ctx, fpm_dtype dt, int64_t b) {
    (void)dt;  // FP32 and FP64 alike (FP64: the update reads the f panels as K segments)
    if (ctx->fuse > 0) return ctx->fuse;
    return (int)std::max<int64_t>(1, std::min<int64_t>(8, 2048 / b));
}

// FP32 scheme of a problem: the option, or auto = F16X3 (three fp16 products,
// 22 significant bits per operand relative to the element itself: FP32-class,
// DESIGN.md Q15).  F16I8 (fp16 main product + int8 cross terms, fixed point
// relative to the row maximum, Q15b) is narrower than FP32 on inputs with a
// large dynamic range, so it is an explicit opt-in only.  F16X3 and F16I8 use
// 2-byte operand halves and per-row / per-column scales; TF32X3 uses 4-byte
// halves and no scales.
SplitScheme scheme_for(const pmm_ctx* ctx, int64_t b) {
    (void)b;
    if (ctx->f32_scheme >= 0) return (SplitScheme)ctx->f32_scheme;
    return SplitScheme::F16X3;
}
bool has_scales(SplitScheme s) { return s != SplitScheme::TF32X3; }
size_t op_bytes(SplitScheme s) { return s == SplitScheme::TF32X3 ? 4 : 2; }

// ---------------------------------------------------------------- setup
// Operand buffers of one slot: receive buffers (NCCL lands pivots in them;
// FP64 copies peers' pivots into them -- FP32 in local / IPC mode stages
// straight from the peers' memory) and the staged operands of a fused update.
void alloc_slot(pmm_ctx* ctx, Device& d, int s) {
    const fpm_dtype dt = ctx->dt;
    const size_t es = esize(dt);
    const size_t op = (dt == FPM_F64) ? 0 : op_bytes(scheme_for(ctx, ctx->b));
    const bool need_recv = ctx->nccl_mode || dt == FPM_F64;
    const size_t fb = (size_t)ctx->fuse_max * ctx->b;  // K of a fused update
    if (need_recv) {
        d.a_recv[s] = dalloc(d, (size_t)d.H * fb * es);  // f panels of H x b
        d.b_recv[s] = dalloc(d, fb * d.W * es);          // f block-rows of b x W
    }
    if (dt == FPM_F64) d.bt[s] = dalloc(d, (size_t)d.W * fb * es);  // W x f b, K-major
    if (dt == FPM_F32) {
        d.a_hi[s] = dalloc(d, (size_t)d.H * fb * op);
        d.a_lo[s] = dalloc(d, (size_t)d.H * fb * op);
        d.b_hi[s] = dalloc(d, (size_t)d.W * fb * op);
        d.b_lo[s] = dalloc(d, (size_t)d.W * fb * op);
        d.sa[s] = static_cast<float*>(dalloc(d, (size_t)d.H * sizeof(float)));
        d.sb[s] = static_cast<float*>(dalloc(d, (size_t)d.W * sizeof(float)));
    }
}

void setup(pmm_ctx* ctx, int64_t N, int64_t b, int p, const colpart_rect* rects, fpm_dtype dt) {
    drop_graph(ctx);
    FPM_CHECK_ARG(dt == FPM_F32 || dt == FPM_F64, "unknown dtype %d", (int)dt);
    FPM_CHECK_ARG(N >= 1 && b >= 1 && N % b == 0, "b must divide N (N=%lld, b=%lld)", (long long)N,
                  (long long)b);
    FPM_CHECK_ARG(dt == FPM_F64 ? b % 8 == 0 : b % 32 == 0, "b must be a multiple of %d",
                  dt == FPM_F64 ? 8 : 32);
    const int expect_p = (ctx->nccl_mode || ctx->ipc_mode) ? ctx->world : (int)ctx->devs.size();
    FPM_CHECK_ARG(p == expect_p, "arrangement has %d devices, context drives %d", p, expect_p);
    FPM_CHECK_ARG(rects != nullptr, "null rects");
    const int64_t n = N / b;
    validate_rects(n, p, rects);

    close_peers(ctx);
    for (auto& d : ctx->devs) free_problem(d);
    ctx->have_problem = false;
    ctx->N = N;
    ctx->b = b;
    ctx->n = n;
    ctx->p = p;
    ctx->dt = dt;
    ctx->rects.assign(rects, rects + p);
    ctx->plan_a.assign(n, {});
    ctx->plan_b.assign(n, {});
    for (int64_t k = 0; k < n; ++k) plan_step(n, p, rects, k, ctx->plan_a[k], ctx->plan_b[k]);

    // Update groups: f consecutive pivots fused into one rank-(f b) update, never
    // across a column boundary (one set of A holders per group) nor a row
    // boundary of any device (one B owner per column per group), so a group's
    // exchange is the plan of its first pivot with longer panels.
    const int f = fuse_factor(ctx, dt, b);
    std::vector<int64_t> cuts;
    for (int q = 0; q < p; ++q)
        if (rects[q].h > 0 && rects[q].w > 0) {
            cuts.push_back(rects[q].col0);
            cuts.push_back(rects[q].row0);
        }
    // Streamed runs (pmm_run) start with two single pivots: the first update
    // waits for only one pivot's panels to cross the host link, and the second
    // group's panels arrive under the first update.
    auto build = [&](std::vector<std::pair<int64_t, int>>& out, int64_t singles) {
        out.clear();
        for (int64_t k = 0; k < n;) {
            int64_t size = std::min<int64_t>(k < singles ? 1 : f, n - k);
            for (int64_t c : cuts)
                if (c > k && c < k + size) size = c - k;
            out.push_back({k, (int)size});
            k += size;
        }
    };
    build(ctx->groups, 0);
    build(ctx->groups_streamed, 2);
    ctx->fuse_max = f;

    const size_t es = esize(dt);
    const bool pinned = has_gpu(ctx);
    for (auto& d : ctx->devs) {
        if (d.cpu) {  // host rectangles; receive buffers for the pivots of one group (two slots)
            d.rect = rects[d.idx];
            d.H = d.rect.h * b;
            d.W = d.rect.w * b;
            if (!d.live()) {
                d.H = d.W = 0;
                continue;
            }
            const size_t HW = (size_t)d.H * d.W;
            d.A = cpu_mem(d, HW * es, pinned);
            d.B = cpu_mem(d, HW * es, pinned);
            d.C = cpu_mem(d, HW * es, false);
            std::memset(d.C, 0, HW * es);
            for (int s = 0; s < 2; ++s) {
                d.h_arecv[s] = cpu_mem(d, (size_t)d.H * f * b * es, pinned);
                d.h_brecv[s] = cpu_mem(d, (size_t)f * b * d.W * es, pinned);
            }
            continue;
        }
        CU(cudaSetDevice(d.cuda_dev));
        d.rect = rects[d.idx];
        d.H = d.rect.h * b;
        d.W = d.rect.w * b;
        for (int s = 0; s < kSlots; ++s) d.b_from[s] = d.idx;
        if (!d.live()) {
            d.H = d.W = 0;
            continue;
        }
        const size_t HW = (size_t)d.H * d.W;
        d.A = dalloc(d, HW * es);
        d.B = dalloc(d, HW * es + 256);  // + the upload-progress flag (IPC peers map it with B)
        d.up_flag = reinterpret_cast<uint64_t*>(static_cast<char*>(d.B) + (HW * es + 63) / 64 * 64);
        CU(cudaMemsetAsync(d.up_flag, 0, 8, d.s_comp));
        d.ooc = d.c_cap > 0 && (int64_t)(HW * es) > d.c_cap;
        if (d.ooc) {  // C_i in pinned host memory, streamed through two band buffers
            d.ring = ring_for(d.c_cap, d.H, d.W, es, ctx->ooc_buffers);
            d.hC = static_cast<float*>(halloc(d, HW * es));
            bp_alloc_bands(d, d.bp, d.ring.R, (size_t)d.ring.rows * d.W * es, (d.H + d.ring.rows - 1) / d.ring.rows);
        } else {
            d.C = dalloc(d, HW * es);
        }
        for (int s = 0; s < 2; ++s) alloc_slot(ctx, d, s);
        if (dt == FPM_F32) {  // in-kernel staging: B column maxima, grid-barrier counters (zeroed)
            d.stg_bmax = static_cast<unsigned*>(dalloc(d, (size_t)d.W * sizeof(unsigned)));
            d.stg_ctr = static_cast<unsigned*>(dalloc(d, 2 * sizeof(unsigned)));
            CU(cudaMemsetAsync(d.stg_ctr, 0, 2 * sizeof(unsigned), d.s_comp));
            CU(cudaMemsetAsync(d.stg_bmax, 0, (size_t)d.W * sizeof(unsigned), d.s_comp));
        }
        for (auto* v : {&d.ev_pack0, &d.ev_pack1, &d.ev_upd0, &d.ev_upd1, &d.ev_up}) {
            v->resize(n);
            for (auto& e : *v) CU(cudaEventCreate(&e));
        }
        if (d.ooc)
            std::memset(d.hC, 0, HW * es);
        else
            CU(cudaMemsetAsync(d.C, 0, HW * es, d.s_comp));
    }

    if (ctx->nccl_mode) {
        // per-column communicators for the vertical B broadcast
        if (ctx->col_comm) {
            nccl().CommDestroy(ctx->col_comm);
            ctx->col_comm = nullptr;
        }
        const colpart_rect& me = rects[ctx->rank];
        const bool live = me.h > 0 && me.w > 0;
        ctx->col_members.clear();
        for (int q = 0; q < p; ++q)
            if (rects[q].h > 0 && rects[q].w > 0 && live && rects[q].col == me.col) ctx->col_members.push_back(q);
        const int color = live ? me.col : NCCL_SPLIT_NOCOLOR;
        ncclConfig_t cfg = nccl_config();
        NC(nccl().CommSplit(ctx->world_comm, color, ctx->rank, &ctx->col_comm, &cfg));
        if (ctx->col_comm) {
            int cn = 0;
            NC(nccl().CommCount(ctx->col_comm, &cn));
            FPM_CHECK_ARG(cn == (int)ctx->col_members.size(), "column communicator has %d ranks, expected %zu", cn,
                          ctx->col_members.size());
        }
    }
    for (auto& d : ctx->devs) {
        if (d.cpu) continue;
        CU(cudaSetDevice(d.cuda_dev));
        CU(cudaDeviceSynchronize());
    }
    ctx->have_problem = true;
}

// ------------------------------------------------------------ iteration parts
ncclDataType_t nccl_dtype(fpm_dtype dt) { return dt == FPM_F64 ? ncclFloat64 : ncclFloat32; }



// Host windows streamed into the resident rectangles during the k-loop
// (pmm_run): block-column k of A and block-row k of B are copied just before
// iteration k needs them, so host->device traffic overlaps earlier updates.
struct HostSrc {
    const void* A;
    const void* B;
    int64_t ld, row_base, col_base;
};

void issue_upload(pmm_ctx* ctx, Device& d, int64_t k, const HostSrc& h) {
    const size_t es = esize(ctx->dt);
    const int64_t b = ctx->b;
    const colpart_rect& r = d.rect;
    CU(cudaSetDevice(d.cuda_dev));
    const int64_t R0 = r.row0 * b - h.row_base, C0 = r.col0 * b - h.col_base;
    if (r.col0 <= k && k < r.col0 + r.w) {
        const int64_t c = k - r.col0;
        const char* src = static_cast<const char*>(h.A) + ((size_t)R0 * h.ld + (size_t)(C0 + c * b)) * es;
        char* dst = static_cast<char*>(d.A) + (size_t)c * d.H * b * es;
        CU(cudaMemcpy2DAsync(dst, b * es, src, h.ld * es, b * es, d.H, cudaMemcpyHostToDevice, d.s_up));
    }
    if (r.row0 <= k && k < r.row0 + r.h) {
        const int64_t rr = k - r.row0;
        const char* src = static_cast<const char*>(h.B) + ((size_t)(R0 + rr * b) * h.ld + (size_t)C0) * es;
        char* dst = static_cast<char*>(d.B) + (size_t)rr * b * d.W * es;
        CU(cudaMemcpy2DAsync(dst, d.W * es, src, h.ld * es, d.W * es, b, cudaMemcpyHostToDevice, d.s_up));
    }
    CU(cudaEventRecord(d.ev_up[k], d.s_up));
    // peers pulling this rank's panels (IPC) and in-kernel staging wait for the
    // flag (after the copies above)
    if (ctx->ipc_mode || ctx->stream_flags)
        if (stream_mem_ops().write64(reinterpret_cast<CUstream>(d.s_up), reinterpret_cast<CUdeviceptr>(d.up_flag),
                                     flag_value(ctx->epoch, k), 0) != CUDA_SUCCESS)
            fail(FPM_ECUDA, "cuStreamWriteValue64 failed");
}

// The comm stream of device d waits until holder / owner q's panels through
// pivot kl have landed (streamed input): q's upload event in one process, q's
// progress flag in peer memory under IPC.
void wait_panels(pmm_ctx* ctx, Device& d, int q, int64_t kl) {
    if (q == d.idx) return;  // own panels: the ev_up wait issued by issue_comm
    if (!ctx->ipc_mode) {
        CU(cudaStreamWaitEvent(d.s_comm, local_dev(ctx, q)->ev_up[kl], 0));
        return;
    }
    if (stream_mem_ops().wait64(reinterpret_cast<CUstream>(d.s_comm), reinterpret_cast<CUdeviceptr>(ctx->peer_flag[q]),
                                flag_value(ctx->epoch, kl), CU_STREAM_WAIT_VALUE_GEQ) != CUDA_SUCCESS)
        fail(FPM_ECUDA, "cuStreamWaitValue64 failed");
}

// Exchange + staging of update group g (pivots k0 .. k0+f-1) on device d's comm
// stream.  All pivots of a group share their holders and owners (setup), so the
// group moves as the plan of k0 with f-times longer panels.
// Fused tail (kFusedSlot): phase 1 merges the group's row / column maxima into
// tmax_a / tmax_b, phase 2 splits it with those maxima into K columns
// [k_off, k_off + f b) of the tail operand (row stride tail_K).  Phase 0: the
// ordinary staging into the slot.
struct TailPhase {
    int phase = 0;
    int64_t k_off = 0;
};

// The B owner of update group g for device d's column, if d may read that
// owner's staged B operand instead of staging its own copy: local FP32 context,
// a double-buffered slot (not the tail), the owner another GPU device on the
// same GPU (its L2 serves the re-reads; peer addresses bypass it).
Device* shared_b_owner(pmm_ctx* ctx, const Device& d, int g, int slot) {
    if (!ctx->share_b || ctx->dt != FPM_F32 || ctx->nccl_mode || ctx->ipc_mode || d.cpu || slot >= 2) return nullptr;
    const int64_t k0 = ctx->groups[g].first;
    for (const Move& m : ctx->plan_b[k0]) {
        if (m.dst != d.idx || m.src == d.idx) continue;
        Device* q = local_dev(ctx, m.src);
        if (q && !q->cpu && q->cuda_dev == d.cuda_dev && q->live() && q->W == d.W) return q;
    }
    return nullptr;
}

int64_t issue_comm(pmm_ctx* ctx, Device& d, int g, int slot, bool first_use, bool streamed,
                   TailPhase tp = TailPhase{}, bool share = false) {
    const size_t es = esize(ctx->dt);
    const int64_t b = ctx->b;
    const int64_t k0 = ctx->groups[g].first;
    const int f = ctx->groups[g].second;
    const int64_t kl = k0 + f - 1;  // last pivot of the group
    const int64_t fb = (int64_t)f * b;
    int64_t bytes = 0;
    CU(cudaSetDevice(d.cuda_dev));
    if (!first_use) CU(cudaStreamWaitEvent(d.s_comm, d.ev_free[slot], 0));
    // shared B operands: this slot's buffers may still be read by the column members
    // whose previous update took its B from here -- wait for those updates too
    if (!first_use && tp.phase == 0 && slot < 2)
        for (auto& q : ctx->devs)
            if (&q != &d && !q.cpu && q.live() && q.b_from[slot] == d.idx)
                CU(cudaStreamWaitEvent(d.s_comm, q.ev_free[slot], 0));
    Device* b_owner = (share && tp.phase == 0) ? shared_b_owner(ctx, d, g, slot) : nullptr;
    if (slot < 2 && tp.phase == 0) d.b_from[slot] = b_owner ? b_owner->idx : d.idx;
    // streamed input: this device's own panels of the group have landed (the
    // upload stream runs ahead, in k order)
    if (streamed) CU(cudaStreamWaitEvent(d.s_comm, d.ev_up[kl], 0));
    const colpart_rect& r = d.rect;

    // FP32 in local / IPC mode: the staging kernels read the pivots straight from
    // the holder's / owner's resident buffer (peer memory over NVLink, or the same
    // GPU), so the transfer is fused into the split -- no receive buffer, no copy.
    const bool fused = ctx->dt == FPM_F32 && !ctx->nccl_mode;
    struct Piece {
        const void* src;        // first pivot's rows; pivot j at src + j * seg_stride
        int64_t seg_stride;     // elements between consecutive pivot panels of the holder
        int64_t row_off, rows;  // in elements (rows of my H x b panels)
    };
    std::vector<Piece> a_pieces;

    // ---- A(rows_i, k0..kl): local if this device's column holds the block-columns
    const bool holder = r.col0 <= k0 && k0 < r.col0 + r.w;
    const void* a_src = nullptr;  // f contiguous H x b panels (holder / received)
    if (holder) {
        a_src = static_cast<const char*>(d.A) + (size_t)(k0 - r.col0) * d.H * b * es;
    } else if (ctx->nccl_mode) {
        a_src = d.a_recv[slot];
    } else {
        for (const Move& m : ctx->plan_a[k0]) {
            if (m.dst != d.idx) continue;
            const colpart_rect& qr = ctx->rects[m.src];
            const int64_t qH = qr.h * b;
            const size_t cnt = (size_t)(m.end - m.begin) * b * b;
            const char* src = static_cast<const char*>(src_A(ctx, m.src)) +
                              ((size_t)(k0 - qr.col0) * qH * b + (size_t)(m.begin - qr.row0) * b * b) * es;
            if (streamed) wait_panels(ctx, d, m.src, kl);
            if (fused) {
                a_pieces.push_back(Piece{src, qH * b, (m.begin - r.row0) * b, (m.end - m.begin) * b});
            } else {  // FP64: copy the f panels' rows into the receive buffer
                for (int j = 0; j < f; ++j) {
                    char* dst = static_cast<char*>(d.a_recv[slot]) +
                                ((size_t)j * d.H * b + (size_t)(m.begin - r.row0) * b * b) * es;
                    CU(cudaMemcpyAsync(dst, src + (size_t)j * qH * b * es, cnt * es, cudaMemcpyDefault, d.s_comm));
                }
                a_src = d.a_recv[slot];
            }
            bytes += (int64_t)(cnt * es) * f;
        }
    }
    // ---- B(k0..kl, cols_i): local if this device's rows hold the block-rows
    const bool owner = r.row0 <= k0 && k0 < r.row0 + r.h;
    const void* b_src = nullptr;  // f b x W rows, contiguous
    if (owner) {
        b_src = static_cast<const char*>(d.B) + (size_t)(k0 - r.row0) * b * d.W * es;
    } else if (ctx->nccl_mode) {
        b_src = d.b_recv[slot];
    } else {
        for (const Move& m : ctx->plan_b[k0]) {
            if (m.dst != d.idx) continue;
            const colpart_rect& orr = ctx->rects[m.src];
            const char* src = static_cast<const char*>(src_B(ctx, m.src)) + (size_t)(k0 - orr.row0) * b * d.W * es;
            if (streamed) wait_panels(ctx, d, m.src, kl);
            if (fused) {
                b_src = src;
            } else {
                CU(cudaMemcpyAsync(d.b_recv[slot], src, (size_t)fb * d.W * es, cudaMemcpyDefault, d.s_comm));
                b_src = d.b_recv[slot];
            }
            bytes += (int64_t)((size_t)fb * d.W * es);
        }
    }
    if (ctx->nccl_mode) {
        const NcclApi& nc = nccl();
        const ncclDataType_t ndt = nccl_dtype(ctx->dt);
        NC(nc.GroupStart());
        for (int j = 0; j < f; ++j) {
            const int64_t k = k0 + j;
            for (const Move& m : ctx->plan_a[k]) {
                if (m.src == m.dst) continue;
                const size_t cnt = (size_t)(m.end - m.begin) * b * b;
                if (m.src == d.idx) {
                    const char* src = static_cast<const char*>(d.A) +
                                      ((size_t)(k - r.col0) * d.H * b + (size_t)(m.begin - r.row0) * b * b) * es;
                    NC(nc.Send(src, cnt, ndt, m.dst, ctx->world_comm, d.s_comm));
                } else if (m.dst == d.idx) {
                    char* dst = static_cast<char*>(d.a_recv[slot]) +
                                ((size_t)j * d.H * b + (size_t)(m.begin - r.row0) * b * b) * es;
                    NC(nc.Recv(dst, cnt, ndt, m.src, ctx->world_comm, d.s_comm));
                    bytes += (int64_t)(cnt * es);
                }
            }
        }
        NC(nc.GroupEnd());
        if (ctx->col_members.size() > 1) {
            int owner_rank = -1;
            for (const Move& m : ctx->plan_b[k0])
                if (m.dst == d.idx) owner_rank = m.src;
            const int root = (int)(std::find(ctx->col_members.begin(), ctx->col_members.end(), owner_rank) -
                                   ctx->col_members.begin());
            void* buf = owner ? const_cast<void*>(b_src) : d.b_recv[slot];
            NC(nc.Broadcast(buf, buf, (size_t)fb * d.W, ndt, root, ctx->col_comm, d.s_comm));
            if (!owner) bytes += (int64_t)((size_t)fb * d.W * es);
        }
    }

    // ---- staging: K-major operands of the fused update (K = f b)
    if (tp.phase != 2) rec_t(d.ev_pack0[g], d.s_comm);
    if (ctx->dt == FPM_F32) {
        const SplitScheme sch = scheme_for(ctx, ctx->b);
        const bool f16 = has_scales(sch);
        const size_t op = op_bytes(sch);
        FPM_CHECK_ARG(b_src != nullptr, "no source of block-row %lld for device %d", (long long)k0, d.idx);
        if (tp.phase == 1) {  // maxima only (TF32X3 has no scales: nothing to do)
            if (f16) {
                d.launches += (a_src ? 1 : (int64_t)a_pieces.size()) + 1;
                if (a_src) {
                    launch_rowmax_seg(static_cast<const float*>(a_src), b, d.H * b, f, d.H, b, d.tmax_a, d.s_comm);
                } else {
                    for (const Piece& pc : a_pieces)
                        launch_rowmax_seg(static_cast<const float*>(pc.src), b, pc.seg_stride, f, pc.rows, b,
                                          d.tmax_a + pc.row_off, d.s_comm);
                }
                launch_colmax(static_cast<const float*>(b_src), d.W, fb, d.W, d.tmax_b, d.s_comm);
            }
        } else {
            const int64_t ld_out = tp.phase == 2 ? d.tail_K : fb;
            const size_t ko = (size_t)tp.k_off * op;
            const unsigned* ga = (tp.phase == 2 && f16) ? d.tmax_a : nullptr;
            const unsigned* gb = (tp.phase == 2 && f16) ? d.tmax_b : nullptr;
            // B rows: maxima, split, scales (F16X3 without given maxima) or the split alone
            d.launches += (a_src ? 1 : (int64_t)a_pieces.size()) + ((f16 && gb == nullptr) ? 3 : 1);
            if (a_src) {  // own or received panels: f consecutive H x b panels
                launch_split_rows_seg(static_cast<const float*>(a_src), b, d.H * b, f, d.H, b, ld_out, sch,
                                      static_cast<char*>(d.a_hi[slot]) + ko, static_cast<char*>(d.a_lo[slot]) + ko,
                                      d.sa[slot], d.s_comm, ga);
            } else {
                for (const Piece& pc : a_pieces)
                    launch_split_rows_seg(
                        static_cast<const float*>(pc.src), b, pc.seg_stride, f, pc.rows, b, ld_out, sch,
                        static_cast<char*>(d.a_hi[slot]) + (size_t)pc.row_off * ld_out * op + ko,
                        static_cast<char*>(d.a_lo[slot]) + (size_t)pc.row_off * ld_out * op + ko,
                        d.sa[slot] + pc.row_off, d.s_comm, ga ? ga + pc.row_off : nullptr);
            }
            if (b_owner) {
                d.launches -= (f16 && gb == nullptr) ? 3 : 1;   // the owner stages this B operand
            } else {
                launch_split_cols(static_cast<const float*>(b_src), d.W, fb, d.W, sch,
                                  static_cast<char*>(d.b_hi[slot]) + ko, static_cast<char*>(d.b_lo[slot]) + ko,
                                  d.sb[slot], d.s_comm, ld_out, gb);
            }
        }
    } else {
        d.a_op[slot] = a_src;  // f panels of H x b, H b apart (own block-columns or the receive buffer)
        launch_transpose_f64(static_cast<const double*>(b_src), d.W, fb, d.W, static_cast<double*>(d.bt[slot]),
                             d.s_comm);
        d.launches += 1;
    }
    if (tp.phase != 2) rec_t(d.ev_pack1[g], d.s_comm);
    if (tp.phase == 0) CU(cudaEventRecord(d.ev_ready[slot], d.s_comm));
    return tp.phase == 2 ? 0 : bytes;
}

// In-kernel staging (option "fused_staging", kernels.hpp StageJob) for device d
// in this k-loop: resident inputs (no host streaming), FP32 F16X3 on the chunked
// kernel (variants 7 / 8, CTA pairs), local or IPC pulls (not NCCL: its
// receives complete on their own schedule), C_i in core, the only GPU device of
// this context on its GPU (the staging warps meet at a grid barrier, so every
// CTA of the update must be resident at once), and a grid of >= 32 CTAs.
bool stream_ops_available() {
    try {
        stream_mem_ops();
        return true;
    } catch (...) {
        return false;
    }
}

// Whether device d's updates on an H x W rectangle stage the next group in
// their staging warps (the kernel / placement / size rules below), FP32 only.
// sampling: every other GPU device of the context on d's GPU counts as sharing
// it (before a problem is set up no device is live; in the run they share it).
bool fused_staging_applies(const pmm_ctx* ctx, const Device& d, int64_t b, int64_t H, int64_t W,
                           bool sampling = false);

bool fused_staging_ok(pmm_ctx* ctx, const Device& d, bool streamed) {
    if (!ctx->fused_staging || ctx->dt != FPM_F32 || ctx->nccl_mode || d.cpu || d.ooc || !d.live()) return false;
    if (streamed && (has_cpu(ctx) || !stream_ops_available())) return false;
    if (!d.stg_bmax || !d.stg_ctr) return false;
    return fused_staging_applies(ctx, d, ctx->b, d.H, d.W);
}

bool fused_staging_applies(const pmm_ctx* ctx, const Device& d, int64_t b, int64_t H, int64_t W, bool sampling) {
    if (!ctx->fused_staging || ctx->nccl_mode || d.cpu || H <= 0 || W <= 0) return false;
    if (scheme_for(ctx, b) != SplitScheme::F16X3 || ctx->cta_group != 2) return false;
    if (!(ctx->kernel_variant == -1 || ctx->kernel_variant == 7 || ctx->kernel_variant == 8 ||
          ctx->kernel_variant == 12 || ctx->kernel_variant == 13))
        return false;
    // every CTA must be resident: alone on the GPU, or confined to its own
    // green partition (devices sharing a GPU under grid caps oversubscribe it).
    // Devices sharing a GPU stage in-kernel only when forced (option value 2):
    // measured on the c4 analogue (eight green partitions, shared B operands)
    // it was no better -- a column owner's update then waits for its members'
    // previous updates before it may stage their shared B -- and worse with
    // the FPM-chosen arrangement (profiles/r02v_fused_staging/hetero_*).
    bool shares_gpu = false;
    for (const auto& q : ctx->devs)
        if (&q != &d && !q.cpu && q.cuda_dev == d.cuda_dev && (sampling || q.live())) shares_gpu = true;
    if (shares_gpu && (!d.green.ctx || ctx->fused_staging != 2)) return false;
    // worth it (option value 1): the two staging warps per CTA must finish well
    // inside the update -- per group (f b of K) they move about (8 H + 12 W) f b
    // bytes while the MMAs take 2 H W f b / (CTAs x ~3 TFLOP/s); at ~4 GB/s per
    // staging warp that is (8 H + 12 W) x kStageCost <= H W (measured crossover,
    // profiles/r02v_fused_staging/fs_crossover.jsonl: off below ~5000^2).  2 forces it on.
    constexpr double kStageCost = 250.0;
    if (ctx->fused_staging == 1 && (8.0 * (double)H + 12.0 * (double)W) * kStageCost > (double)H * (double)W)
        return false;
    const int64_t tiles = ((H + 255) / 256) * ((W + 255) / 256);
    return std::min<int64_t>(d.num_sms / 2, tiles) >= 1;
}

// The upload-progress flag of device q as device d reads it (own / local
// device memory, or the IPC peer mapping).
const unsigned long long* flag_of(pmm_ctx* ctx, const Device& d, int q) {
    if (q == d.idx) return reinterpret_cast<const unsigned long long*>(d.up_flag);
    if (ctx->ipc_mode) return reinterpret_cast<const unsigned long long*>(ctx->peer_flag[q]);
    return reinterpret_cast<const unsigned long long*>(local_dev(ctx, q)->up_flag);
}

// The staging of update group g into operand slot `slot` of device d as a job
// for the previous update's staging warp: the same sources as issue_comm's
// FP32 local / IPC path (own panels, or the holders' / owner's resident memory;
// streamed: after their progress flags show the group's panels landed).
// Returns the pivot bytes pulled from other devices; job.active = 0 when the
// group has more A pieces than a job holds.
int64_t build_stage_job(pmm_ctx* ctx, const Device& d, int g, int slot, StageJob& J, bool streamed, bool with_b) {
    const int64_t b = ctx->b;
    const int64_t k0 = ctx->groups[g].first;
    const int f = ctx->groups[g].second;
    const int64_t fb = (int64_t)f * b;
    const colpart_rect& r = d.rect;
    int64_t bytes = 0;
    J = StageJob{};
    J.nseg = f;
    J.K = b;
    J.lda = b;
    J.ld_out = fb;
    auto wait_for = [&](int q) {
        if (!streamed) return;
        const unsigned long long* fl = flag_of(ctx, d, q);
        for (int i = 0; i < J.nwait; ++i)
            if (J.wait_flag[i] == fl) return;
        J.wait_flag[J.nwait++] = fl;
    };
    if (r.col0 <= k0 && k0 < r.col0 + r.w) {  // own block-columns: f panels of H x b
        J.a[0] = StagePiece{static_cast<const float*>(d.A) + (size_t)(k0 - r.col0) * d.H * b, d.H * b, 0, d.H};
        J.npieces = 1;
        wait_for(d.idx);
    } else {
        for (const Move& m : ctx->plan_a[k0]) {
            if (m.dst != d.idx) continue;
            if (J.npieces == kMaxStagePieces) return 0;
            const colpart_rect& qr = ctx->rects[m.src];
            const int64_t qH = qr.h * b;
            const float* src = static_cast<const float*>(src_A(ctx, m.src)) +
                               ((size_t)(k0 - qr.col0) * qH * b + (size_t)(m.begin - qr.row0) * b * b);
            J.a[J.npieces++] = StagePiece{src, qH * b, (m.begin - r.row0) * b, (m.end - m.begin) * b};
            wait_for(m.src);
            bytes += (m.end - m.begin) * b * b * 4 * f;
        }
    }
    if (!with_b) {  // B: the column owner's staged operand (share_b)
    } else if (r.row0 <= k0 && k0 < r.row0 + r.h) {
        J.b_src = static_cast<const float*>(d.B) + (size_t)(k0 - r.row0) * b * d.W;
        wait_for(d.idx);
    } else {
        for (const Move& m : ctx->plan_b[k0]) {
            if (m.dst != d.idx) continue;
            const colpart_rect& orr = ctx->rects[m.src];
            J.b_src = static_cast<const float*>(src_B(ctx, m.src)) + (size_t)(k0 - orr.row0) * b * d.W;
            wait_for(m.src);
            bytes += fb * d.W * 4;
        }
    }
    J.need = streamed ? flag_value(ctx->epoch, k0 + f - 1) : 0;
    if (J.npieces == 0 || (with_b && J.b_src == nullptr)) return 0;
    J.ldb = d.W;
    J.Kb = fb;
    J.W = d.W;
    J.a_hi = d.a_hi[slot];
    J.a_lo = d.a_lo[slot];
    J.sa = d.sa[slot];
    J.b_hi = d.b_hi[slot];
    J.b_lo = d.b_lo[slot];
    J.sb = d.sb[slot];
    J.bmax = d.stg_bmax;
    J.ctr = d.stg_ctr;
    J.active = 1;
    return bytes;
}

// FP32 update of group g from operand slot `slot` over all of C_i.
UpdateArgs f32_args(pmm_ctx* ctx, const Device& d, int g, int slot) {
    UpdateArgs a;
    a.a_hi = d.a_hi[slot];
    a.a_lo = d.a_lo[slot];
    // the B operand: this device's, or the column owner's on the same GPU (share_b)
    const Device* bd = (slot < 2 && d.b_from[slot] != d.idx) ? local_dev(ctx, d.b_from[slot]) : &d;
    a.bt_hi = bd->b_hi[slot];
    a.bt_lo = bd->b_lo[slot];
    const SplitScheme sch = scheme_for(ctx, ctx->b);
    const bool f16 = has_scales(sch);
    a.sa = f16 ? d.sa[slot] : nullptr;
    a.sb = f16 ? bd->sb[slot] : nullptr;
    a.C = static_cast<float*>(d.C);
    a.M = d.H;
    a.Nc = d.W;
    a.K = (int64_t)ctx->groups[g].second * ctx->b;
    a.ldc = d.W;
    a.scheme = sch;
    a.cta_group = ctx->cta_group;
    a.num_sms = d.num_sms;
    a.accumulate = ctx->groups[g].first != 0;  // the first update writes C = A(0..) B(0..): no zeroing, no read of C
    a.raster_group = raster_group_for(ctx, d, sch);
    a.l2_hint_b = ctx->l2_hint_b;
    a.variant = ctx->kernel_variant;  // -1: auto (F16X3 / TF32X3: variant 8; F16I8: 6)
    a.chunk_k = ctx->chunk_k;
    a.raster_snake = ctx->raster_snake != 0;
    // NCCL kernels need shared memory to co-run with the persistent update:
    // F16I8 then takes variant 5 (198 KB) instead of 6 (224 KB); F16X3's auto variant 8 uses 160 KB
    if (a.variant < 0 && ctx->nccl_mode && sch == SplitScheme::F16I8) a.variant = 5;
    return a;
}

// The same update restricted to rows [r0, r0 + m) of C_i, written to `Cband`
// (row stride W): rows r0.. of the A operand and of its scales.
UpdateArgs band_args(const UpdateArgs& a, int64_t r0, int64_t m, float* Cband) {
    const size_t op = op_bytes(a.scheme);
    UpdateArgs x = a;
    x.a_hi = static_cast<const char*>(a.a_hi) + (size_t)r0 * a.K * op;
    x.a_lo = static_cast<const char*>(a.a_lo) + (size_t)r0 * a.K * op;
    x.sa = a.sa ? a.sa + r0 : nullptr;
    x.C = Cband;
    x.M = m;
    return x;
}

void issue_update(pmm_ctx* ctx, Device& d, int g, int slot, const StageJob* next = nullptr,
                  bool staged_in_kernel = false) {
    const int64_t k0 = ctx->groups[g].first;
    const int f = ctx->groups[g].second;
    CU(cudaSetDevice(d.cuda_dev));
    if (staged_in_kernel) {  // update g - 1 staged this group on this stream: nothing to wait for
        rec_t(d.ev_pack0[g], d.s_comp);
        rec_t(d.ev_pack1[g], d.s_comp);
    } else {
        CU(cudaStreamWaitEvent(d.s_comp, d.ev_ready[slot], 0));
    }
    if (ctx->dt == FPM_F32 && slot < 2 && d.b_from[slot] != d.idx)  // the owner staged this update's B
        CU(cudaStreamWaitEvent(d.s_comp, local_dev(ctx, d.b_from[slot])->ev_ready[slot], 0));
    rec_t(d.ev_upd0[g], d.s_comp);
    // out-of-core band order: reversed every other update, the last two
    // bands kept on the device between updates (option "ooc_keep")
    BandCall bc;
    bc.accumulate = k0 != 0;
    bc.reverse = ctx->ooc_keep && (g & 1);
    bc.kept_head = ctx->ooc_keep && g > 0;
    bc.keep_tail = ctx->ooc_keep && g + 1 < (int)ctx->groups.size();
    if (ctx->dt == FPM_F32) {
        UpdateArgs a = f32_args(ctx, d, g, slot);
        if (next) a.stage = *next;
        if (d.ooc) {
            // out of core: the same update, one row band of C_i at a time (rows
            // r0.. of the A operand and its scales, the band buffer as C)
            d.launches += banded_update(d.bp, d.ring, reinterpret_cast<char*>(d.hC), d.H, (size_t)d.W * 4, bc,
                                        d.s_comp, [&](int64_t r0, int64_t m, void* band) {
                                            launch_update_f32(band_args(a, r0, m, static_cast<float*>(band)),
                                                              d.s_comp);
                                        });
        } else {
            launch_update_f32(a, d.s_comp);
            d.launches += 1;
        }
    } else {
        // FP64: the group's f panels (H x b each, H b apart) as K segments of one
        // rank-(f b) update against the transposed block-rows (W x f b)
        const double* aop = static_cast<const double*>(d.a_op[slot]);
        const int64_t b = ctx->b, K = (int64_t)f * b;
        if (d.ooc) {
            d.launches += banded_update(d.bp, d.ring, reinterpret_cast<char*>(d.hC), d.H, (size_t)d.W * 8, bc,
                                        d.s_comp, [&](int64_t r0, int64_t m, void* band) {
                                            launch_update_f64(aop + (size_t)r0 * b, b,
                                                              static_cast<const double*>(d.bt[slot]),
                                                              static_cast<double*>(band), m, d.W, K, d.W, k0 != 0,
                                                              d.num_sms, d.s_comp, b, d.H * b);
                                        });
        } else {
            launch_update_f64(aop, b, static_cast<const double*>(d.bt[slot]), static_cast<double*>(d.C), d.H, d.W, K,
                              d.W, k0 != 0, d.num_sms, d.s_comp, b, d.H * b);
            d.launches += 1;
        }
    }
    rec_t(d.ev_upd1[g], d.s_comp);
    CU(cudaEventRecord(d.ev_free[slot], d.s_comp));
}

// The N/b iterations.  Iteration 0 writes C_i = A(0) B(0), so C needs no
// zeroing.  With `host` set, the pivot panels are streamed from host memory one
// iteration ahead of their use (pmm_run).
// Host destination of C for compute_into / pmm_run.
struct HostDst {
    void* C;
    int64_t ld, row_base, col_base;
};

// Groups of the download-overlapped tail (option "e2e_tail"; FP32, resident
// C_i).  Auto: enough of the last updates to cover the device -> host copy of
// C_i -- per element of C_i the copy costs 4 B at ~55 GB/s, the k-loop 2 N flop
// at ~3 TFLOP/s per SM (measured) -- but, when the inputs are streamed in
// (pmm_run), no more than leaves the uploads (8 B per element of C_i) under the
// groups before the tail: the tail's staging needs its pivots on the device.
//
// Band-streamed tail (one device, pmm_run, `tail_stream`): the tail needs its B
// rows (4 B per element of C_i) before it starts and its A rows only band by
// band, so the uploads under the groups before the tail are 8 B per element for
// those groups plus 4 B for the tail's B: X (4 u + 4 u) + (1 - X) 4 u <= X c,
// i.e. the non-tail fraction X >= r / (1 - r), r = 4 u / c.
bool streamed_tail_ok(const pmm_ctx* ctx);
int tail_groups(pmm_ctx* ctx, bool streamed) {
    const int G = (int)ctx->groups.size();
    if (ctx->dt != FPM_F32 || ctx->e2e_tail == 0 || G == 0) return 0;
    if (ctx->e2e_tail > 0) return std::min({ctx->e2e_tail, G, kMaxTail});
    const double rate_per_sm = scheme_for(ctx, ctx->b) == SplitScheme::F16I8 ? 3.9e12 : 3.0e12;  // measured, c5
    double r = 0.0;
    for (auto& d : ctx->devs)
        if (d.live() && !d.ooc && !d.cpu)
            r = std::max(r, (4.0 / 55e9) / (2.0 * (double)ctx->N / (rate_per_sm * d.num_sms)));
    if (r == 0.0) return 0;
    // host link slower than the updates (r >= 0.5, e.g. N = 16384 on one B200):
    // the band-streamed tail takes the whole k-loop -- all of B's rows first,
    // then A's rows band by band, each band's C leaving over the other PCIe
    // direction while the next band's rows arrive -- so the step is about the
    // H2D bytes plus one band, instead of H2D plus most of the D2H
    if (streamed && streamed_tail_ok(ctx) && r >= 0.5) return std::min(G, kMaxTail);
    int L = (int)std::ceil(G * 1.05 * r);
    if (streamed && streamed_tail_ok(ctx) && r < 0.5)  // 0.55: the tail may start somewhat late (measured, c5:
        L = std::min(L, (int)std::floor(G * (1.0 - 0.55 * r / (1.0 - r))));  // L = 12 of 25 best, 8: -4 %, 16: -8 %)
    else if (streamed)
        L = std::min(L, G - (int)std::ceil(G * 2.0 * r));
    return std::max(1, std::min({L, G, kMaxTail}));
}

// Operand slots 2 .. 2+L-1 for the tail groups (allocated once per problem).
void ensure_tail_slots(pmm_ctx* ctx, Device& d, int L) {
    CU(cudaSetDevice(d.cuda_dev));
    for (; d.tail_slots < L; ++d.tail_slots) alloc_slot(ctx, d, 2 + d.tail_slots);
}

// The tail as ONE operand (local / IPC FP32): the pivots of groups gt.. staged
// side by side along K with common F16X3 row / column scales, so each band of
// C_i takes one update of K = tail_K -- one read-modify-write of the band
// instead of one per group.  The same sum per element as the group-major
// loop, with one scale per row over the tail instead of one per group.
bool use_fused_tail(const pmm_ctx* ctx) { return ctx->tail_fuse && ctx->dt == FPM_F32 && !ctx->nccl_mode; }
// One device holding the whole problem (p = 1, local): its tail operand can be
// staged from rows that arrive band by band.
bool streamed_tail_ok(const pmm_ctx* ctx) {
    return ctx->tail_stream && use_fused_tail(ctx) && !ctx->ipc_mode && ctx->devs.size() == 1 && !ctx->devs[0].cpu &&
           ctx->devs[0].live() && !ctx->devs[0].ooc && ctx->devs[0].rect.h * ctx->b == ctx->N &&
           ctx->devs[0].rect.w * ctx->b == ctx->N;
}

void ensure_fused_tail(pmm_ctx* ctx, Device& d, int gt, bool rows) {
    int64_t K = 0;
    for (size_t g = gt; g < ctx->groups.size(); ++g) K += (int64_t)ctx->groups[g].second * ctx->b;
    d.tail_K = K;
    if (K <= d.tail_K_alloc && (d.tail_rows != nullptr || !rows)) return;
    CU(cudaSetDevice(d.cuda_dev));
    CU(cudaDeviceSynchronize());
    for (void* p : d.tail_allocs) cudaFree(p);
    d.tail_allocs.clear();
    const size_t op = op_bytes(scheme_for(ctx, ctx->b));
    auto get = [&](size_t bytes) {
        void* p = nullptr;
        if (cudaMalloc(&p, bytes) != cudaSuccess) {
            cudaGetLastError();
            fail(FPM_ENOMEM, "device %d: cannot allocate %zu bytes for the fused tail", d.cuda_dev, bytes);
        }
        d.tail_allocs.push_back(p);
        return p;
    };
    const int s = kFusedSlot;
    d.a_hi[s] = get((size_t)d.H * K * op);
    d.a_lo[s] = get((size_t)d.H * K * op);
    d.b_hi[s] = get((size_t)d.W * K * op);
    d.b_lo[s] = get((size_t)d.W * K * op);
    d.sa[s] = static_cast<float*>(get((size_t)d.H * sizeof(float)));
    d.sb[s] = static_cast<float*>(get((size_t)d.W * sizeof(float)));
    d.tmax_a = static_cast<unsigned*>(get((size_t)d.H * sizeof(unsigned)));
    d.tmax_b = static_cast<unsigned*>(get((size_t)d.W * sizeof(unsigned)));
    d.tail_rows = rows ? static_cast<float*>(get((size_t)d.H * K * sizeof(float))) : nullptr;
    d.tail_K_alloc = K;
}

// The tail of the k-loop, band-major: for each band of C_i rows, the updates of
// the L tail groups (slots 2..), then its device -> host copy on the copy
// stream -- band j's copy overlaps the updates of bands j+1.., so only the last
// band's copy is exposed.  The same sums in the same order per element as the
// group-major loop (each element still receives the groups in k order).
// Row bands of the tail: whole bands of `band` rows (multiples of 256, the
// CTA-pair tile rows), the last one halved down to 256 rows (band, ..., band/2,
// band/4, ..., 256, 256) so the copy left exposed after the last update is
// small; the copy stream keeps pace with the updates, so earlier bands' copies
// finish under the following bands.
std::vector<std::pair<int64_t, int64_t>> tail_bands(int64_t H, int64_t band) {
    std::vector<std::pair<int64_t, int64_t>> out;
    int64_t r0 = 0;
    while (H - r0 > band) {
        out.push_back({r0, band});
        r0 += band;
    }
    int64_t rest = H - r0;  // <= band: halve it while the halves stay >= 256 rows
    while (rest > 512) {
        const int64_t half = (rest / 2 + 255) / 256 * 256;
        out.push_back({r0, half});
        r0 += half;
        rest -= half;
    }
    if (rest > 0) out.push_back({r0, rest});
    return out;
}

void issue_tail(pmm_ctx* ctx, Device& d, int g0, int L, const HostDst& out) {
    CU(cudaSetDevice(d.cuda_dev));
    const bool fused = d.tail_fused_run;
    if (fused) {
        CU(cudaStreamWaitEvent(d.s_comp, d.ev_ready[kFusedSlot], 0));
    } else {
        for (int t = 0; t < L; ++t) CU(cudaStreamWaitEvent(d.s_comp, d.ev_ready[2 + t], 0));
    }
    CU(cudaEventRecord(d.ev_upd0[g0], d.s_comp));
    UpdateArgs fa;  // fused: all tail pivots in one operand of K = tail_K
    if (fused) {
        fa = f32_args(ctx, d, g0, kFusedSlot);
        fa.K = d.tail_K;
    }
    const int64_t b = ctx->b;
    const int64_t R0 = d.rect.row0 * b - out.row_base, C0 = d.rect.col0 * b - out.col_base;
    float* C = static_cast<float*>(d.C);
    for (const auto& bd : tail_bands(d.H, ctx->tail_band)) {
        const int64_t r0 = bd.first, m = bd.second;
        if (fused) {
            launch_update_f32(band_args(fa, r0, m, C + (size_t)r0 * d.W), d.s_comp);
            d.launches += 1;
        }
        for (int t = 0; t < L && !fused; ++t) {
            const UpdateArgs a = f32_args(ctx, d, g0 + t, 2 + t);
            launch_update_f32(band_args(a, r0, m, C + (size_t)r0 * d.W), d.s_comp);
            d.launches += 1;
        }
        CU(cudaEventRecord(d.bp.done[0], d.s_comp));
        if (r0 + m >= d.H) CU(cudaEventRecord(d.ev_io0, d.s_comp));  // last band updated
        CU(cudaStreamWaitEvent(d.bp.s_d2h, d.bp.done[0], 0));
        char* dst = static_cast<char*>(out.C) + ((size_t)(R0 + r0) * out.ld + (size_t)C0) * 4;
        CU(cudaMemcpy2DAsync(dst, out.ld * 4, C + (size_t)r0 * d.W, d.W * 4, d.W * 4, m, cudaMemcpyDeviceToHost,
                             d.bp.s_d2h));
    }
    CU(cudaEventRecord(d.ev_upd1[g0], d.s_comp));
    for (int t = 1; t < L; ++t) {  // the tail's time is booked on its first group
        CU(cudaEventRecord(d.ev_upd0[g0 + t], d.s_comp));
        CU(cudaEventRecord(d.ev_upd1[g0 + t], d.s_comp));
    }
    if (fused) {
        CU(cudaEventRecord(d.ev_free[kFusedSlot], d.s_comp));
    } else {
        for (int t = 0; t < L; ++t) CU(cudaEventRecord(d.ev_free[2 + t], d.s_comp));
    }
    CU(cudaEventRecord(d.ev_io1, d.bp.s_d2h));  // C_i in host memory
}

// The N/b iterations.  Iteration 0 writes C_i = A(0) B(0), so C needs no
// zeroing.  With `host` set, the pivot panels are streamed from host memory one
// iteration ahead of their use (pmm_run).  With `out` set, C_i is also copied
// to host memory, overlapped with the last updates where possible (tail);
// returns true for each device whose copy was done here (tail_done).
void issue_kloop(pmm_ctx* ctx, const HostSrc* host, const HostDst* out, int L, int64_t* bytes_out);
void capture_kloop(pmm_ctx* ctx);
void finish_kloop(pmm_ctx* ctx, pmm_stats* st, bool streamed, const std::vector<char>* tail_done, int64_t bytes,
                  int64_t launches);

// ------------------------------------------------------------ CPU devices
// The k-loop of a host-CPU device (P:15's iteration on a socket, P:18 kernel):
// per update group, gather A(rows_i, k0..kl) and B(k0..kl, cols_i) into host
// receive buffers -- pieces held by GPU devices are pulled device -> host on
// this device's pull streams, pieces of CPU devices copied -- then
// C_i (+)= A B with the team's GEMM.  The next group's pulls are issued before
// the current GEMM (two slots), so they overlap it.  Pivot sources are resident
// inputs that the loop never writes, so no ordering with the GPU streams is
// needed (pmm_compute's inputs are resident before it starts).
void cpu_kloop(pmm_ctx* ctx, Device& d) {
    using clk = std::chrono::steady_clock;
    const auto t_begin = clk::now();
    const int G = (int)ctx->groups.size();
    const size_t es = esize(ctx->dt);
    const int64_t b = ctx->b;
    const colpart_rect& r = d.rect;
    d.cpu_pack_s.assign(G, 0.0);
    d.cpu_upd_s.assign(G, 0.0);
    d.cpu_bytes = 0;
    struct Op {
        const void* A = nullptr;
        int64_t seg_stride = 0;  // A: f panels of H x b (row stride b), seg_stride apart
        const void* B = nullptr; // B: f b rows of W
        std::vector<cudaStream_t> wait;
    };
    auto secs = [](clk::time_point a, clk::time_point z) { return std::chrono::duration<double>(z - a).count(); };
    auto gather = [&](int g, int slot) {
        const auto t0 = clk::now();
        Op op;
        const int64_t k0 = ctx->groups[g].first;
        const int f = ctx->groups[g].second;
        auto copy = [&](void* dst, const void* src, size_t bytes, const Device* q) {
            if (q->cpu) {
                std::memcpy(dst, src, bytes);
            } else {
                cudaStream_t st = pull_stream(d, q->cuda_dev);
                CU(cudaSetDevice(q->cuda_dev));
                CU(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, st));
                if (std::find(op.wait.begin(), op.wait.end(), st) == op.wait.end()) op.wait.push_back(st);
            }
            d.cpu_bytes += (int64_t)bytes;
        };
        if (r.col0 <= k0 && k0 < r.col0 + r.w) {  // own block-columns
            op.A = static_cast<const char*>(d.A) + (size_t)(k0 - r.col0) * d.H * b * es;
        } else {
            for (const Move& m : ctx->plan_a[k0]) {
                if (m.dst != d.idx) continue;
                const Device* q = local_dev(ctx, m.src);
                const colpart_rect& qr = ctx->rects[m.src];
                const int64_t qH = qr.h * b;
                const size_t cnt = (size_t)(m.end - m.begin) * b * b * es;
                const char* src = static_cast<const char*>(q->A) +
                                  ((size_t)(k0 - qr.col0) * qH * b + (size_t)(m.begin - qr.row0) * b * b) * es;
                for (int j = 0; j < f; ++j)
                    copy(static_cast<char*>(d.h_arecv[slot]) + ((size_t)j * d.H * b + (size_t)(m.begin - r.row0) * b * b) * es,
                         src + (size_t)j * qH * b * es, cnt, q);
            }
            op.A = d.h_arecv[slot];
        }
        op.seg_stride = d.H * b;
        if (r.row0 <= k0 && k0 < r.row0 + r.h) {  // own block-rows
            op.B = static_cast<const char*>(d.B) + (size_t)(k0 - r.row0) * b * d.W * es;
        } else {
            for (const Move& m : ctx->plan_b[k0]) {
                if (m.dst != d.idx) continue;
                const Device* q = local_dev(ctx, m.src);
                const colpart_rect& orr = ctx->rects[m.src];
                copy(d.h_brecv[slot], static_cast<const char*>(q->B) + (size_t)(k0 - orr.row0) * b * d.W * es,
                     (size_t)f * b * d.W * es, q);
                op.B = d.h_brecv[slot];
            }
        }
        FPM_CHECK_ARG(op.B != nullptr, "no source of block-row %lld for CPU device %d", (long long)k0, d.idx);
        d.cpu_pack_s[g] += secs(t0, clk::now());
        return op;
    };
    auto wait = [&](const Op& op) {
        for (cudaStream_t st : op.wait) CU(cudaStreamSynchronize(st));
    };
    Op cur = gather(0, 0);
    wait(cur);
    for (int g = 0; g < G; ++g) {
        Op nxt;
        if (g + 1 < G) nxt = gather(g + 1, (g + 1) & 1);  // pulls of the next group under this GEMM
        const int64_t K = (int64_t)ctx->groups[g].second * b;
        const bool acc = ctx->groups[g].first != 0;  // the first update writes C_i = A(0..) B(0..)
        const auto t0 = clk::now();
        if (ctx->dt == FPM_F32)
            cpu::gemm_f32(d.team, d.H, d.W, K, static_cast<const float*>(cur.A), b, b, cur.seg_stride,
                          static_cast<const float*>(cur.B), d.W, static_cast<float*>(d.C), d.W, acc);
        else
            cpu::gemm_f64(d.team, d.H, d.W, K, static_cast<const double*>(cur.A), b, b, cur.seg_stride,
                          static_cast<const double*>(cur.B), d.W, static_cast<double*>(d.C), d.W, acc);
        d.cpu_upd_s[g] = secs(t0, clk::now());
        if (g + 1 < G) {
            wait(nxt);
            cur = nxt;
        }
    }
    d.cpu_loop_s = secs(t_begin, clk::now());
}

// Runs every live CPU device's k-loop on a thread of its own for the lifetime
// of the object; join() waits and re-throws the first failure.
struct CpuLoops {
    std::vector<std::thread> threads;
    std::vector<std::exception_ptr> errs;
    explicit CpuLoops(pmm_ctx* ctx) {
        size_t n = 0;
        for (auto& d : ctx->devs) n += (d.cpu && d.live()) ? 1 : 0;
        errs.assign(n, nullptr);  // sized before any thread holds a pointer into it
        size_t i = 0;
        for (auto& d : ctx->devs) {
            if (!d.cpu || !d.live()) continue;
            Device* dp = &d;
            std::exception_ptr* e = &errs[i++];
            threads.emplace_back([ctx, dp, e] {
                try {
                    cpu_kloop(ctx, *dp);
                } catch (...) {
                    *e = std::current_exception();
                }
            });
        }
    }
    void join() {
        for (auto& t : threads)
            if (t.joinable()) t.join();
        for (auto& e : errs)
            if (e) std::rethrow_exception(e);
    }
    ~CpuLoops() {
        for (auto& t : threads)
            if (t.joinable()) t.join();
    }
};

void compute(pmm_ctx* ctx, pmm_stats* st, const HostSrc* host = nullptr, const HostDst* out = nullptr,
             std::vector<char>* tail_done = nullptr) {
    if (!ctx->have_problem) fail(FPM_ESTATE, "pmm_compute before pmm_setup");
    if (ctx->ipc_mode && !ctx->peers_ready)
        fail(FPM_ESTATE, "IPC context: pmm_ipc_import must follow pmm_setup before pmm_compute");
    if (host) ++ctx->epoch;  // this run's progress-flag values (IPC: every rank in step)
    // streamed input: the grouping that starts with single pivots (setup)
    struct GroupSwap {
        pmm_ctx* c;
        bool on;
        GroupSwap(pmm_ctx* c_, bool on_) : c(c_), on(on_) {
            if (on) std::swap(c->groups, c->groups_streamed);
        }
        ~GroupSwap() {
            if (on) std::swap(c->groups, c->groups_streamed);
        }
    } group_swap(ctx, host != nullptr);
    const int L = out ? tail_groups(ctx, host != nullptr) : 0;
    if (tail_done) tail_done->assign(ctx->devs.size(), 0);
    for (size_t i = 0; i < ctx->devs.size(); ++i) {
        Device& d = ctx->devs[i];
        d.tail_fused_run = false;
        d.tail_streamed_run = false;
        if (L > 0 && d.live() && !d.ooc && !d.cpu) {
            // before the timed region (cudaMalloc synchronises)
            if (use_fused_tail(ctx)) {
                const bool rows = host != nullptr && streamed_tail_ok(ctx);
                ensure_fused_tail(ctx, d, (int)ctx->groups.size() - L, rows);
                d.tail_fused_run = true;
                d.tail_streamed_run = rows;
            } else {
                ensure_tail_slots(ctx, d, L);
            }
            if (tail_done) (*tail_done)[i] = 1;
        }
    }
    int64_t launches0 = 0;
    for (auto& d : ctx->devs) {
        launches0 += d.launches;
        d.bp.bytes = 0;
    }
    for (auto& d : ctx->devs) {
        if (!d.live() || d.cpu) continue;
        CU(cudaSetDevice(d.cuda_dev));
        CU(cudaStreamSynchronize(d.s_comp));
        CU(cudaStreamSynchronize(d.s_comm));
    }
    // pmm_compute on resident inputs: the whole k-loop is one CUDA graph,
    // captured on first use and replayed (option "graph")
    // (not with green partitions: measured, replays lose the per-device SM
    // confinement -- c4 analogue 0.37 s replayed vs 0.23 s issued eagerly)
    const bool use_graph = ctx->graph && !host && !out && !ctx->nccl_mode && !ctx->sm_partition && !has_cpu(ctx);
    FPM_CHECK_ARG(!(host && has_cpu(ctx)), "streamed host input with CPU devices (pmm_run uploads first)");
    // CPU devices run their k-loops on their own threads, concurrently with the
    // GPU devices' streams (their pivots come from resident buffers only)
    CpuLoops cpu_loops(ctx);
    int64_t bytes = 0, launches = 0;
    if (use_graph) {
        if (!ctx->gexec) capture_kloop(ctx);
        Device& d0 = ctx->devs[0];
        CU(cudaSetDevice(d0.cuda_dev));
        CU(cudaGraphLaunch(ctx->gexec, d0.s_comp));
        bytes = ctx->g_bytes;
        launches = ctx->g_launches;
        for (auto& d : ctx->devs) d.bp.bytes = d.g_ooc_bytes;
    } else {
        issue_kloop(ctx, host, out, L, &bytes);
        launches = -launches0;
        for (auto& d : ctx->devs) launches += d.launches;
    }
    cpu_loops.join();
    finish_kloop(ctx, st, host != nullptr, tail_done, bytes, launches);
}

// Everything from ev_start to ev_stop of one k-loop, on the devices' streams.
// Band-streamed fused tail (pmm_run with one device holding all of A, B and C;
// option "tail_stream").  Every element of C needs the last pivot, so no band of
// C can leave before the tail's pivots arrived -- but a band needs only ITS rows
// of the tail's A panels.  So the tail's B rows (one copy) are uploaded first,
// then its A rows band by band into `tail_rows` (H x tail_K, row-major: one 2D
// copy per band); B is staged once, each band's A rows as they land, and band
// j's update and device -> host copy start as soon as its rows are staged: the
// D2H of early bands overlaps the H2D of later ones.  Same operand, scales
// (per-row over the tail's K, per-column over its rows) and sums as the fused
// tail of issue_tail.
void issue_tail_streamed(pmm_ctx* ctx, Device& d, int gt, const HostSrc& h, const HostDst& out) {
    const int64_t b = ctx->b;
    const int64_t kt = ctx->groups[gt].first;  // first tail pivot
    const int64_t K = d.tail_K;
    FPM_CHECK_ARG(kt * b + K == ctx->N && d.tail_rows != nullptr, "streamed tail: inconsistent tail");
    const SplitScheme sch = scheme_for(ctx, b);
    const size_t op = op_bytes(sch);
    const colpart_rect& r = d.rect;
    CU(cudaSetDevice(d.cuda_dev));
    const auto bands = tail_bands(d.H, ctx->tail_band);
    while (d.ev_band_up.size() < bands.size()) {
        cudaEvent_t e1, e2;
        CU(cudaEventCreateWithFlags(&e1, cudaEventDisableTiming));
        CU(cudaEventCreateWithFlags(&e2, cudaEventDisableTiming));
        d.ev_band_up.push_back(e1);
        d.ev_band_st.push_back(e2);
    }
    if (!d.ev_tail_b) CU(cudaEventCreateWithFlags(&d.ev_tail_b, cudaEventDisableTiming));
    const int64_t R0 = r.row0 * b - h.row_base, C0 = r.col0 * b - h.col_base;
    // uploads (behind the non-tail groups' on s_up): the tail's B rows, then A by bands
    {
        const char* src = static_cast<const char*>(h.B) + ((size_t)(R0 + kt * b) * h.ld + (size_t)C0) * 4;
        char* dst = static_cast<char*>(d.B) + (size_t)kt * b * d.W * 4;
        CU(cudaMemcpy2DAsync(dst, d.W * 4, src, h.ld * 4, d.W * 4, K, cudaMemcpyHostToDevice, d.s_up));
        CU(cudaEventRecord(d.ev_tail_b, d.s_up));
    }
    for (size_t j = 0; j < bands.size(); ++j) {
        const int64_t r0 = bands[j].first, m = bands[j].second;
        const char* src = static_cast<const char*>(h.A) + ((size_t)(R0 + r0) * h.ld + (size_t)(C0 + kt * b)) * 4;
        CU(cudaMemcpy2DAsync(d.tail_rows + (size_t)r0 * K, K * 4, src, h.ld * 4, K * 4, m, cudaMemcpyHostToDevice,
                             d.s_up));
        CU(cudaEventRecord(d.ev_band_up[j], d.s_up));
    }
    for (int64_t k = kt; k < ctx->n; ++k) CU(cudaEventRecord(d.ev_up[k], d.s_up));  // every tail pivot landed
    // staging on the comm stream: B once (column maxima over the tail's rows), then A band by band
    // (the tail groups' own staging events stay empty: the staging is booked on ev_tpack0..1)
    for (int g = gt; g < (int)ctx->groups.size(); ++g) {
        rec_t(d.ev_pack0[g], d.s_comm);
        rec_t(d.ev_pack1[g], d.s_comm);
    }
    rec_t(d.ev_tpack0, d.s_comm);
    CU(cudaStreamWaitEvent(d.s_comm, d.ev_tail_b, 0));
    launch_split_cols(static_cast<const float*>(d.B) + (size_t)kt * b * d.W, d.W, K, d.W, sch, d.b_hi[kFusedSlot],
                      d.b_lo[kFusedSlot], d.sb[kFusedSlot], d.s_comm, K, nullptr);
    d.launches += has_scales(sch) ? 3 : 1;
    CU(cudaEventRecord(d.ev_ready[kFusedSlot], d.s_comm));
    for (size_t j = 0; j < bands.size(); ++j) {
        const int64_t r0 = bands[j].first, m = bands[j].second;
        CU(cudaStreamWaitEvent(d.s_comm, d.ev_band_up[j], 0));
        launch_split_rows_seg(d.tail_rows + (size_t)r0 * K, K, 0, 1, m, K, K, sch,
                              static_cast<char*>(d.a_hi[kFusedSlot]) + (size_t)r0 * K * op,
                              static_cast<char*>(d.a_lo[kFusedSlot]) + (size_t)r0 * K * op,
                              d.sa[kFusedSlot] ? d.sa[kFusedSlot] + r0 : nullptr, d.s_comm, nullptr);
        d.launches += 1;
        CU(cudaEventRecord(d.ev_band_st[j], d.s_comm));
    }
    rec_t(d.ev_tpack1, d.s_comm);
    // updates band by band, each band's copy to the host right after its update
    CU(cudaStreamWaitEvent(d.s_comp, d.ev_ready[kFusedSlot], 0));
    CU(cudaEventRecord(d.ev_upd0[gt], d.s_comp));
    UpdateArgs fa = f32_args(ctx, d, gt, kFusedSlot);
    fa.K = K;
    fa.accumulate = kt != 0;  // the groups before the tail wrote C (none: the tail is the whole k-loop)
    const int64_t oR0 = r.row0 * b - out.row_base, oC0 = r.col0 * b - out.col_base;
    float* C = static_cast<float*>(d.C);
    for (size_t j = 0; j < bands.size(); ++j) {
        const int64_t r0 = bands[j].first, m = bands[j].second;
        CU(cudaStreamWaitEvent(d.s_comp, d.ev_band_st[j], 0));
        launch_update_f32(band_args(fa, r0, m, C + (size_t)r0 * d.W), d.s_comp);
        d.launches += 1;
        CU(cudaEventRecord(d.bp.done[0], d.s_comp));
        if (r0 + m >= d.H) CU(cudaEventRecord(d.ev_io0, d.s_comp));  // last band updated
        CU(cudaStreamWaitEvent(d.bp.s_d2h, d.bp.done[0], 0));
        char* dst = static_cast<char*>(out.C) + ((size_t)(oR0 + r0) * out.ld + (size_t)oC0) * 4;
        CU(cudaMemcpy2DAsync(dst, out.ld * 4, C + (size_t)r0 * d.W, d.W * 4, d.W * 4, m, cudaMemcpyDeviceToHost,
                             d.bp.s_d2h));
    }
    CU(cudaEventRecord(d.ev_upd1[gt], d.s_comp));
    for (int g = gt + 1; g < (int)ctx->groups.size(); ++g) {  // the tail's time is booked on its first group
        CU(cudaEventRecord(d.ev_upd0[g], d.s_comp));
        CU(cudaEventRecord(d.ev_upd1[g], d.s_comp));
    }
    CU(cudaEventRecord(d.ev_free[kFusedSlot], d.s_comp));
    CU(cudaEventRecord(d.ev_io1, d.bp.s_d2h));  // C_i in host memory
}

void issue_kloop(pmm_ctx* ctx, const HostSrc* host, const HostDst* out, int L, int64_t* bytes_out) {
    const int ngroups = (int)ctx->groups.size();
    const int gt = ngroups - L;  // first tail group
    for (auto& d : ctx->devs) {
        if (d.cpu) continue;
        CU(cudaSetDevice(d.cuda_dev));
        rec_t(d.ev_start, d.s_comp);
        if (!g_capturing) {  // (a capture forks every stream from its origin instead)
            CU(cudaStreamWaitEvent(d.s_comm, d.ev_start, 0));
            CU(cudaStreamWaitEvent(d.s_up, d.ev_start, 0));
        }
    }
    const bool streamed = host != nullptr;
    int64_t bytes = 0;
    // tail devices take tail groups from slots 2.. and update them band-major
    // after the loop; everyone else (and every group before gt) as usual
    auto in_tail = [&](const Device& d, int g) { return g >= gt && d.live() && !d.ooc && !d.cpu; };
    auto slot_of = [&](const Device& d, int g) {
        return in_tail(d, g) ? (d.tail_fused_run ? kFusedSlot : 2 + (g - gt)) : (g & 1);
    };
    // band-streamed tail: its uploads, staging and updates are issued after the loop
    auto streamed_tail = [&](const Device& d, int g) { return in_tail(d, g) && d.tail_streamed_run; };
    // in-kernel staging: group g >= 1 (not in the tail) was staged by update g - 1
    ctx->stream_flags = false;
    for (auto& d : ctx->devs) {
        d.fs_run = fused_staging_ok(ctx, d, streamed);
        ctx->stream_flags = ctx->stream_flags || (d.fs_run && streamed);
    }
    auto staged_in_kernel = [&](const Device& d, int g) { return d.fs_run && g >= 1 && !in_tail(d, g); };
    std::vector<char> job_ok(ctx->devs.size(), 0);  // the previous update carried this group's job
    for (int g = 0; g < ngroups; ++g) {
        const int64_t k0 = ctx->groups[g].first;
        if (streamed)
            for (int64_t k = k0; k < k0 + ctx->groups[g].second; ++k)
                for (auto& d : ctx->devs)
                    if (d.live() && !d.cpu && !streamed_tail(d, g)) issue_upload(ctx, d, k, *host);
        if (ctx->nccl_mode) {
            // every rank takes part in the NCCL calls, live or not
            Device& d = ctx->devs[0];
            if (d.live()) {
                const int slot = slot_of(d, g);
                bytes += issue_comm(ctx, d, g, slot, g < 2 && slot < 2, streamed);
                if (!in_tail(d, g)) issue_update(ctx, d, g, slot);
            } else {
                NC(nccl().GroupStart());
                NC(nccl().GroupEnd());
            }
            continue;
        }
        for (size_t di = 0; di < ctx->devs.size(); ++di) {
            Device& d = ctx->devs[di];
            if (d.live() && !d.cpu && !streamed_tail(d, g) && !(staged_in_kernel(d, g) && job_ok[di])) {
                const int slot = slot_of(d, g);
                if (in_tail(d, g) && d.tail_fused_run) {  // fused tail, pass 1: merge the maxima
                    if (g == gt) {
                        CU(cudaMemsetAsync(d.tmax_a, 0, (size_t)d.H * sizeof(unsigned), d.s_comm));
                        CU(cudaMemsetAsync(d.tmax_b, 0, (size_t)d.W * sizeof(unsigned), d.s_comm));
                    }
                    bytes += issue_comm(ctx, d, g, slot, false, streamed, TailPhase{1, 0});
                } else {
                    bytes += issue_comm(ctx, d, g, slot, g < 2 && slot < 2, streamed, TailPhase{}, g < gt);
                }
            }
        }
        // the updates of group g, each carrying the staging of group g + 1 for
        // its device (in-kernel staging).  With shared B operands (share_b,
        // green partitions of one GPU) a column member's job stages its A rows
        // only: it reads the B operand the owner's update stages, whose launch
        // first waits for the members' updates that read its previous B in that
        // slot (the b_from values of the slot's previous use).
        const int nx = g + 1, sx = nx & 1;
        const size_t nd = ctx->devs.size();
        std::vector<StageJob> jobs(nd);
        std::vector<int64_t> job_bytes(nd, 0);
        std::vector<int> owner_of(nd, -1);  // device index whose B this device's update nx reads
        for (size_t di = 0; di < nd; ++di) {
            Device& d = ctx->devs[di];
            if (!d.live() || d.cpu || in_tail(d, g) || !d.fs_run || nx >= ngroups || in_tail(d, nx)) continue;
            const Device* ow = shared_b_owner(ctx, d, nx, sx);
            if (ow && !ow->fs_run) continue;  // the owner stages eagerly: so does this member (issue_comm)
            job_bytes[di] = build_stage_job(ctx, d, nx, sx, jobs[di], streamed, ow == nullptr);
            owner_of[di] = ow ? ow->idx : d.idx;
        }
        for (size_t di = 0; di < nd; ++di) {  // a member's job needs the owner's (B) job
            if (!jobs[di].active || owner_of[di] == ctx->devs[di].idx) continue;
            for (size_t oi = 0; oi < nd; ++oi)
                if (ctx->devs[oi].idx == owner_of[di] && !jobs[oi].active) jobs[di].active = 0;
        }
        for (size_t di = 0; di < nd; ++di) {
            Device& d = ctx->devs[di];
            if (!d.live() || d.cpu || in_tail(d, g)) continue;
            const bool here = staged_in_kernel(d, g) && job_ok[di];
            const StageJob& job = jobs[di];
            const bool stages_b = job.active && job.b_src != nullptr;
            if (stages_b && nx >= 2) {  // readers of this device's B in slot sx at group nx - 2
                CU(cudaSetDevice(d.cuda_dev));
                for (auto& q : ctx->devs)
                    if (&q != &d && !q.cpu && q.live() && q.b_from[sx] == d.idx)
                        CU(cudaStreamWaitEvent(d.s_comp, q.ev_free[sx], 0));
            }
            issue_update(ctx, d, g, g & 1, job.active ? &job : nullptr, here);
            if (stages_b) CU(cudaEventRecord(d.ev_ready[sx], d.s_comp));  // members' update nx waits for it
            job_ok[di] = job.active ? 1 : 0;
            if (job.active) bytes += job_bytes[di];
        }
        for (size_t di = 0; di < nd; ++di)
            if (jobs[di].active) ctx->devs[di].b_from[sx] = owner_of[di];
    }
    // fused tail, pass 2: split every tail group with the merged maxima into its
    // K range of the tail operand
    for (auto& d : ctx->devs) {
        if (L == 0 || !d.live() || d.ooc || d.cpu || !d.tail_fused_run || d.tail_streamed_run) continue;
        CU(cudaSetDevice(d.cuda_dev));
        rec_t(d.ev_tpack0, d.s_comm);
        int64_t k_off = 0;
        for (int g = gt; g < ngroups; ++g) {
            issue_comm(ctx, d, g, kFusedSlot, false, streamed, TailPhase{2, k_off});
            k_off += (int64_t)ctx->groups[g].second * ctx->b;
        }
        rec_t(d.ev_tpack1, d.s_comm);
        CU(cudaEventRecord(d.ev_ready[kFusedSlot], d.s_comm));
    }
    if (L > 0)
        for (auto& d : ctx->devs) {
            if (!d.live() || d.ooc || d.cpu) continue;
            if (d.tail_streamed_run) issue_tail_streamed(ctx, d, gt, *host, *out);
            else issue_tail(ctx, d, gt, L, *out);
        }
    for (auto& d : ctx->devs) {
        if (d.cpu) continue;
        CU(cudaSetDevice(d.cuda_dev));
        if (d.ooc) bp_join(d.bp, d.s_comp);  // C_i is complete once its last band is back in host memory
        rec_t(d.ev_stop, d.s_comp);
    }
    *bytes_out = bytes;
}

// Capture one k-loop into ctx->gexec: every stream of every device is forked
// from device 0's compute stream and joined back into it.
void capture_kloop(pmm_ctx* ctx) {
    Device& d0 = ctx->devs[0];
    for (auto& d : ctx->devs) {  // the graph starts from a clean band pipeline
        d.bp.used[0] = false;
        for (int i = 0; i < kMaxBandBufs; ++i) d.bp.used[i] = false;
        std::fill(d.bp.band_used.begin(), d.bp.band_used.end(), 0);
        d.bp.last = d.bp.last_step = -1;
        d.bp.next = 0;
        d.bp.dir = 1;
        d.bp.bytes = 0;
    }
    int64_t launches0 = 0;
    for (auto& d : ctx->devs) launches0 += d.launches;
    CU(cudaSetDevice(d0.cuda_dev));
    if (!ctx->ev_fork) CU(cudaEventCreateWithFlags(&ctx->ev_fork, cudaEventDisableTiming));
    const cudaStream_t origin = d0.s_comp;
    CU(cudaStreamBeginCapture(origin, cudaStreamCaptureModeRelaxed));
    int64_t bytes = 0;
    try {
        CU(cudaEventRecord(ctx->ev_fork, origin));
        for (auto& d : ctx->devs) {
            CU(cudaSetDevice(d.cuda_dev));
            for (cudaStream_t s : {d.s_comp, d.s_comm, d.bp.s_h2d, d.bp.s_d2h})
                if (s != origin) CU(cudaStreamWaitEvent(s, ctx->ev_fork, 0));
        }
        g_capturing = true;
        issue_kloop(ctx, nullptr, nullptr, 0, &bytes);
        g_capturing = false;
        for (auto& d : ctx->devs) {
            CU(cudaSetDevice(d.cuda_dev));
            int j = 0;
            for (cudaStream_t s : {d.s_comp, d.s_comm, d.bp.s_h2d, d.bp.s_d2h}) {
                if (s == origin) continue;
                CU(cudaEventRecord(d.ev_join[j], s));
                CU(cudaSetDevice(d0.cuda_dev));
                CU(cudaStreamWaitEvent(origin, d.ev_join[j], 0));
                CU(cudaSetDevice(d.cuda_dev));
                ++j;
            }
        }
    } catch (...) {
        g_capturing = false;
        cudaGraph_t junk = nullptr;
        cudaSetDevice(d0.cuda_dev);
        cudaStreamEndCapture(origin, &junk);
        if (junk) cudaGraphDestroy(junk);
        cudaGetLastError();
        throw;
    }
    CU(cudaSetDevice(d0.cuda_dev));
    cudaGraph_t graph = nullptr;
    CU(cudaStreamEndCapture(origin, &graph));
    cudaError_t e = cudaGraphInstantiate(&ctx->gexec, graph, 0);
    cudaGraphDestroy(graph);
    if (e != cudaSuccess) {
        ctx->gexec = nullptr;
        fail(FPM_ECUDA, "cudaGraphInstantiate: %s", cudaGetErrorString(e));
    }
    ctx->g_bytes = bytes;
    ctx->g_launches = -launches0;
    for (auto& d : ctx->devs) {
        ctx->g_launches += d.launches;
        d.g_ooc_bytes = d.bp.bytes;
    }
}

// Wait for the k-loop and fill the statistics.
void finish_kloop(pmm_ctx* ctx, pmm_stats* st, bool streamed, const std::vector<char>* tail_done, int64_t bytes,
                  int64_t launches) {
    const int ngroups = (int)ctx->groups.size();
    double t_max = 0.0, t_tail_copy = 0.0;
    std::vector<double> span(ctx->devs.size(), 0.0);
    for (size_t i = 0; i < ctx->devs.size(); ++i) {
        Device& d = ctx->devs[i];
        if (d.cpu) {
            if (d.live()) t_max = std::max(t_max, d.cpu_loop_s);
            if (d.live()) span[i] = d.cpu_loop_s;
            bytes += d.live() ? d.cpu_bytes : 0;
            continue;
        }
        CU(cudaSetDevice(d.cuda_dev));
        if (ctx->nccl_mode) {  // poll the communicators while waiting (the last
            nccl_wait(ctx, d.ev_stop);  // update waited for the last exchange)
        } else if (ctx->ipc_mode) {
            ipc_wait(d.ev_stop);
        } else {
            CU(cudaEventSynchronize(d.ev_stop));
        }
        CU(cudaStreamSynchronize(d.s_comm));
        span[i] = d.live() ? (double)elapsed_ms(d.ev_start, d.ev_stop) * 1e-3 : 0.0;
        t_max = std::max(t_max, (double)elapsed_ms(d.ev_start, d.ev_stop) * 1e-3);
        if (tail_done && (*tail_done)[i]) {  // copy still draining after the last update
            CU(cudaEventSynchronize(d.ev_io1));
            // exposed copy: from the end of the last band's updates (a timing event
            // recorded before its copy is issued) to the end of that copy
            t_tail_copy = std::max(t_tail_copy, std::max(0.0, (double)elapsed_ms(d.ev_io0, d.ev_io1) * 1e-3));
        }
    }
    if (st) {
        std::memset(st, 0, sizeof(*st));
        st->t_compute_s = t_max;
        st->t_download_s = t_tail_copy;
        if (streamed) {
            double tu = 0.0;  // until the last host->device panel landed
            for (auto& d : ctx->devs)
                if (d.live() && !d.cpu) tu = std::max(tu, (double)elapsed_ms(d.ev_start, d.ev_up[ctx->n - 1]) * 1e-3);
            st->t_upload_s = tu;
        }
        st->iters = ctx->n;
        st->updates = ngroups;
        for (auto& d : ctx->devs)
            if (d.ooc) {
                if (d.idx < 63) st->ooc_devices |= (int64_t)1 << d.idx;
                st->ooc_bytes += d.bp.bytes;
            }
        st->comm_bytes = bytes;
        st->kernel_launches = launches;
        st->gflops = t_max > 0 ? 2.0 * (double)ctx->N * (double)ctx->N * (double)ctx->N / t_max * 1e-9 : 0.0;
        double mx = 0.0, sum = 0.0;
        int cnt = 0;
        for (auto& d : ctx->devs) {
            if (!d.live()) continue;
            double comp = 0.0, upd = 0.0;
            for (int g = 0; g < ngroups && d.cpu; ++g) {  // host-timed gather + GEMM of each group
                comp += d.cpu_pack_s[g] + d.cpu_upd_s[g];
                upd += d.cpu_upd_s[g];
            }
            for (int g = 0; g < ngroups && !d.cpu; ++g) {
                const double u = elapsed_ms(d.ev_upd0[g], d.ev_upd1[g]) * 1e-3;
                comp += u + elapsed_ms(d.ev_pack0[g], d.ev_pack1[g]) * 1e-3;
                upd += u;
            }
            if (d.tail_fused_run && !d.cpu) comp += elapsed_ms(d.ev_tpack0, d.ev_tpack1) * 1e-3;
            if (d.idx < FPM_MAX_DEVICES) {
                st->per_dev_compute_s[d.idx] = comp;
                st->per_dev_update_s[d.idx] = upd;
            }
            mx = std::max(mx, comp);
            sum += comp;
            ++cnt;
        }
        st->imbalance = (cnt > 0 && sum > 0) ? mx / (sum / cnt) - 1.0 : 0.0;
        for (size_t i = 0; i < ctx->devs.size(); ++i)
            if (ctx->devs[i].idx < FPM_MAX_DEVICES) st->per_dev_span_s[ctx->devs[i].idx] = span[i];
    }
}

// ------------------------------------------------------------ host transfers
void copy_rows(void* dst, size_t dpitch, const void* src, size_t spitch, size_t width, int64_t rows) {
    for (int64_t r = 0; r < rows; ++r)
        std::memcpy(static_cast<char*>(dst) + (size_t)r * dpitch, static_cast<const char*>(src) + (size_t)r * spitch,
                    width);
}

void check_window(pmm_ctx* ctx, const Device& d, int64_t ld, int64_t row_base, int64_t col_base) {
    const int64_t R0 = d.rect.row0 * ctx->b, C0 = d.rect.col0 * ctx->b;
    FPM_CHECK_ARG(row_base >= 0 && col_base >= 0 && R0 >= row_base && C0 >= col_base &&
                      C0 - col_base + d.W <= ld,
                  "device %d rectangle outside the host window (ld=%lld)", d.idx, (long long)ld);
}

void upload(pmm_ctx* ctx, const void* A, const void* B, int64_t ld, int64_t row_base, int64_t col_base,
            double* t_out) {
    if (!ctx->have_problem) fail(FPM_ESTATE, "pmm_upload before pmm_setup");
    FPM_CHECK_ARG(A && B, "null host matrix");
    const size_t es = esize(ctx->dt);
    const int64_t b = ctx->b;
    double t = 0.0;
    for (auto& d : ctx->devs) {
        if (!d.live()) continue;
        check_window(ctx, d, ld, row_base, col_base);
        const int64_t R0 = d.rect.row0 * b - row_base, C0 = d.rect.col0 * b - col_base;
        if (d.cpu) {  // host to host: block-column panels of A, rows of B
            for (int64_t c = 0; c < d.rect.w; ++c)
                copy_rows(static_cast<char*>(d.A) + (size_t)c * d.H * b * es, b * es,
                          static_cast<const char*>(A) + ((size_t)R0 * ld + (size_t)(C0 + c * b)) * es, ld * es, b * es,
                          d.H);
            copy_rows(d.B, d.W * es, static_cast<const char*>(B) + ((size_t)R0 * ld + (size_t)C0) * es, ld * es,
                      d.W * es, d.H);
            std::memset(d.C, 0, (size_t)d.H * d.W * es);
            continue;
        }
        CU(cudaSetDevice(d.cuda_dev));
        CU(cudaEventRecord(d.ev_io0, d.s_comp));
        for (int64_t c = 0; c < d.rect.w; ++c) {
            const char* src = static_cast<const char*>(A) + ((size_t)R0 * ld + (size_t)(C0 + c * b)) * es;
            char* dst = static_cast<char*>(d.A) + (size_t)c * d.H * b * es;
            CU(cudaMemcpy2DAsync(dst, b * es, src, ld * es, b * es, d.H, cudaMemcpyHostToDevice, d.s_comp));
        }
        const char* srcB = static_cast<const char*>(B) + ((size_t)R0 * ld + (size_t)C0) * es;
        CU(cudaMemcpy2DAsync(d.B, d.W * es, srcB, ld * es, d.W * es, d.H, cudaMemcpyHostToDevice, d.s_comp));
        if (!d.ooc) CU(cudaMemsetAsync(d.C, 0, (size_t)d.H * d.W * es, d.s_comp));
        CU(cudaEventRecord(d.ev_io1, d.s_comp));
    }
    for (auto& d : ctx->devs) {
        if (!d.live() || d.cpu) continue;
        CU(cudaSetDevice(d.cuda_dev));
        CU(cudaEventSynchronize(d.ev_io1));
        t = std::max(t, (double)elapsed_ms(d.ev_io0, d.ev_io1) * 1e-3);
    }
    if (t_out) *t_out = t;
}

void download(pmm_ctx* ctx, void* C, int64_t ld, int64_t row_base, int64_t col_base, double* t_out,
              const std::vector<char>* skip = nullptr) {
    if (!ctx->have_problem) fail(FPM_ESTATE, "pmm_download before pmm_setup");
    FPM_CHECK_ARG(C, "null host matrix");
    const size_t es = esize(ctx->dt);
    const int64_t b = ctx->b;
    double t = 0.0;
    std::vector<char> copied(ctx->devs.size(), 0);
    for (size_t i = 0; i < ctx->devs.size(); ++i) {
        Device& d = ctx->devs[i];
        if (!d.live() || (skip && (*skip)[i])) continue;
        check_window(ctx, d, ld, row_base, col_base);
        const int64_t R0 = d.rect.row0 * b - row_base, C0 = d.rect.col0 * b - col_base;
        char* dst = static_cast<char*>(C) + ((size_t)R0 * ld + (size_t)C0) * es;
        if (d.cpu) {
            copy_rows(dst, ld * es, d.C, d.W * es, d.W * es, d.H);
            continue;
        }
        copied[i] = 1;
        CU(cudaSetDevice(d.cuda_dev));
        CU(cudaEventRecord(d.ev_io0, d.s_comp));
        if (d.ooc) {  // C_i already in host memory (compute joined its band copies)
            CU(cudaStreamSynchronize(d.bp.s_d2h));
            copy_rows(dst, ld * es, d.hC, d.W * es, d.W * es, d.H);
        } else {
            CU(cudaMemcpy2DAsync(dst, ld * es, d.C, d.W * es, d.W * es, d.H, cudaMemcpyDeviceToHost, d.s_comp));
        }
        CU(cudaEventRecord(d.ev_io1, d.s_comp));
    }
    for (size_t i = 0; i < ctx->devs.size(); ++i) {
        Device& d = ctx->devs[i];
        if (!copied[i]) continue;
        CU(cudaSetDevice(d.cuda_dev));
        CU(cudaEventSynchronize(d.ev_io1));
        t = std::max(t, (double)elapsed_ms(d.ev_io0, d.ev_io1) * 1e-3);
    }
    if (t_out) *t_out = t;
}

void fill_synthetic(pmm_ctx* ctx, uint64_t seed_a, uint64_t seed_b, int dist) {
    if (!ctx->have_problem) fail(FPM_ESTATE, "pmm_fill_synthetic before pmm_setup");
    const size_t es = esize(ctx->dt);
    const bool f64 = ctx->dt == FPM_F64;
    const int64_t b = ctx->b;
    for (auto& d : ctx->devs) {
        if (!d.live()) continue;
        const int64_t R0 = d.rect.row0 * b, C0 = d.rect.col0 * b;
        if (d.cpu) {  // the same counter-based generator on the host
            for (int64_t c = 0; c < d.rect.w; ++c)
                cpu::fill_synthetic(d.team, static_cast<char*>(d.A) + (size_t)c * d.H * b * es, f64, b, seed_a, ctx->N,
                                    R0, C0 + c * b, d.H, b, dist);
            cpu::fill_synthetic(d.team, d.B, f64, d.W, seed_b, ctx->N, R0, C0, d.H, d.W, dist);
            std::memset(d.C, 0, (size_t)d.H * d.W * es);
            continue;
        }
        CU(cudaSetDevice(d.cuda_dev));
        for (int64_t c = 0; c < d.rect.w; ++c)
            launch_fill_synthetic(static_cast<char*>(d.A) + (size_t)c * d.H * b * es, f64, b, seed_a, ctx->N, R0,
                                  C0 + c * b, d.H, b, dist, d.s_comp);
        launch_fill_synthetic(d.B, f64, d.W, seed_b, ctx->N, R0, C0, d.H, d.W, dist, d.s_comp);
        if (!d.ooc) CU(cudaMemsetAsync(d.C, 0, (size_t)d.H * d.W * es, d.s_comp));
    }
    for (auto& d : ctx->devs) {
        if (!d.live() || d.cpu) continue;
        CU(cudaSetDevice(d.cuda_dev));
        CU(cudaStreamSynchronize(d.s_comp));
    }
}

// ------------------------------------------------------------ speed sampling
double t975(int df) {
    static const double tab[] = {0,      12.706, 4.303, 3.182, 2.776, 2.571, 2.447, 2.365, 2.306, 2.262, 2.228,
                                 2.201, 2.179,  2.160, 2.145, 2.131, 2.120, 2.110, 2.101, 2.093, 2.086};
    if (df <= 20) return tab[df < 1 ? 1 : df];
    if (df <= 30) return 2.086 + (2.042 - 2.086) * (df - 20) / 10.0;
    if (df <= 60) return 2.042 + (2.000 - 2.042) * (df - 30) / 30.0;
    return 1.96;
}

// P:9 "The speed function of the application can be built more efficiently by
// timing this kernel"; P:10 (iii) "experiments are repeated multiple times
// until the results are statistically reliable"; P:18 kernel Ci += A(b) x B(b)
// on sqrt(x) x sqrt(x) submatrices.  Speed = 2 x b^3 flop / time (Q7, Q8).
//
// dev = -1 samples every device of the context at the same time (P:10 (ii):
// "Processes are synchronised ... ensures that the resources will be shared
// between the maximum number of processes"), which captures the contention of
// devices emulated on one GPU; each repetition launches the kernel on all
// devices and times each on its own stream.  Outputs are then p x nsizes.
// Side of each sample size x = m^2 blocks (P:18 sqrt(x) x sqrt(x) submatrices).
std::vector<int64_t> sample_sides(const int64_t* sizes, int nsizes) {
    std::vector<int64_t> ms(nsizes);
    for (int j = 0; j < nsizes; ++j) {
        const int64_t x = sizes[j];
        FPM_CHECK_ARG(x >= 1, "size must be >= 1");
        int64_t m = (int64_t)std::llround(std::sqrt((double)x));
        while (m * m > x) --m;
        while ((m + 1) * (m + 1) <= x) ++m;
        FPM_CHECK_ARG(m * m == x, "size %lld is not a perfect square (P:18 sqrt(x) x sqrt(x))", (long long)x);
        ms[j] = m;
    }
    return ms;
}

// Sample shapes: h x w blocks (C is h b x w b); the square sizes of fpm_sample
// are m x m, fpm_sample_rects takes any rectangle (the speed "does not
// vary with the nearly square shapes"; the operating-point refinement samples
// the rectangles the arrangement gave each device, reading Q26).
struct Shape {
    int64_t h, w;
};

// One CPU device's sampling kernel: C (h b x w b) += A (h b x f b) B (f b x w b)
// -- the k-loop's fused update -- on all c cores of the device at once, each on
// h b / c rows ("the speed of a socket executing the ACML kernels
// simultaneously on c cores, with the problem size x / c on each core"
// (ii) synchronised cores), host-timed (the synchronous approach).
struct CpuRunner {
    Device* d;
    fpm_dtype dt;
    int64_t b, fb, Hm = 0, Wm = 0;
    void *A = nullptr, *B = nullptr, *C = nullptr;
    CpuRunner(pmm_ctx* ctx, Device* dev, fpm_dtype dt_, int64_t b_, const std::vector<Shape>& shp)
        : d(dev), dt(dt_), b(b_), fb((int64_t)fuse_factor(ctx, dt_, b_) * b_) {
        int64_t area = 0;
        for (const Shape& x : shp) {
            Hm = std::max(Hm, x.h * b);
            Wm = std::max(Wm, x.w * b);
            area = std::max(area, x.h * x.w * b * b);
        }
        const size_t es = esize(dt);
        auto get = [&](void*& p, size_t bytes) {
            if (posix_memalign(&p, 64, std::max<size_t>(bytes, 64)) != 0) fail(FPM_ENOMEM, "host allocation failed");
        };
        get(A, (size_t)Hm * fb * es);
        get(B, (size_t)fb * Wm * es);
        get(C, (size_t)area * es);
        cpu::fill_synthetic(d->team, A, dt == FPM_F64, fb, 101, std::max(Hm, Wm), 0, 0, Hm, fb, FPM_DIST_PM1);
        cpu::fill_synthetic(d->team, B, dt == FPM_F64, Wm, 102, std::max(Hm, Wm), 0, 0, fb, Wm, FPM_DIST_PM1);
        std::memset(C, 0, (size_t)area * es);
    }
    ~CpuRunner() {
        std::free(A);
        std::free(B);
        std::free(C);
    }
    double flops(const Shape& x) const { return 2.0 * (double)(x.h * x.w) * (double)b * (double)b * (double)fb; }
    // one run, completed on return
    void run(const Shape& x) {
        const int64_t Mx = x.h * b, Nx = x.w * b;
        if (dt == FPM_F32)
            cpu::gemm_f32(d->team, Mx, Nx, fb, static_cast<const float*>(A), fb, fb, 0, static_cast<const float*>(B),
                          Wm, static_cast<float*>(C), Nx, true);
        else
            cpu::gemm_f64(d->team, Mx, Nx, fb, static_cast<const double*>(A), fb, fb, 0,
                          static_cast<const double*>(B), Wm, static_cast<double*>(C), Nx, true);
    }
};

// One GPU device's sampling kernel, as the k-loop runs it: staging (split /
// transpose) of an f-pivot group and the fused rank-(f b) update on an h b x w b
// C; shapes whose C exceeds the device's C cap run out of core through the band
// ring in the k-loop's steady state (bands kept, order reversed).  Where
// the k-loop stages the next group inside the update (§4.8, same rule), so
// does the sampler: each run's update reads one operand set and its staging
// warps split the panels into the other for the next run, so the timed kernel
// carries the staging the run pays (hidden, not added).
struct GpuRunner {
    pmm_ctx* ctx;
    Device* d;
    fpm_dtype dt;
    int64_t b, fb;
    size_t es, op;
    SplitScheme sch;
    Device mem;          // owns the allocations (and the band pipeline of out-of-core sizes)
    char* hC = nullptr;  // pinned host C for sizes above the device's C cap
    void *C = nullptr, *Ap = nullptr, *Bp = nullptr, *Bt = nullptr;
    void *ah = nullptr, *al = nullptr, *bh = nullptr, *bl = nullptr;
    float *sa = nullptr, *sb = nullptr;
    int64_t Hm = 0, Wm = 0;  // largest rows / columns of C over this device's shapes
    int runs = 0;            // runs at the current size (out-of-core band order alternates)
    // in-kernel staging: a second operand set, the staging warps' scratch, and
    // the shape each set currently holds
    void *ah2 = nullptr, *al2 = nullptr, *bh2 = nullptr, *bl2 = nullptr;
    float *sa2 = nullptr, *sb2 = nullptr;
    unsigned *bmax = nullptr, *ctr = nullptr;
    int cur = 0;
    int64_t held[2][2] = {{-1, -1}, {-1, -1}};

    bool ooc_at(int64_t Mx, int64_t Nx) const { return d->c_cap > 0 && (int64_t)(Mx * Nx * es) > d->c_cap; }
    Ring ring_at(int64_t Mx, int64_t Nx) const { return ring_for(d->c_cap, Mx, Nx, es, ctx->ooc_buffers); }
    double flops(const Shape& x) const { return 2.0 * (double)(x.h * x.w) * (double)b * (double)b * (double)fb; }

    GpuRunner(pmm_ctx* c, Device* dev, fpm_dtype dt_, int64_t b_, const std::vector<Shape>& shp)
        : ctx(c), d(dev), dt(dt_), b(b_), fb((int64_t)fuse_factor(c, dt_, b_) * b_), es(dt_ == FPM_F64 ? 8 : 4),
          op(op_bytes(scheme_for(c, b_))), sch(scheme_for(c, b_)) {
        mem.cuda_dev = d->cuda_dev;
        CU(cudaSetDevice(d->cuda_dev));
        int64_t in_area = 0, out_area = 0, nbands = 0;
        size_t band_bytes = 0;
        for (const Shape& x : shp) {
            const int64_t Mx = x.h * b, Nx = x.w * b;
            Hm = std::max(Hm, Mx);
            Wm = std::max(Wm, Nx);
            if (!ooc_at(Mx, Nx)) {
                in_area = std::max(in_area, Mx * Nx);
                continue;
            }
            out_area = std::max(out_area, Mx * Nx);
            const int64_t rows = ring_at(Mx, Nx).rows;
            nbands = std::max(nbands, (Mx + rows - 1) / rows);
            band_bytes = std::max(band_bytes, (size_t)rows * Nx * es);
        }
        C = dalloc(mem, (size_t)in_area * es);
        if (out_area > 0) {
            bp_init(mem.bp);
            hC = static_cast<char*>(halloc(mem, (size_t)out_area * es));
            std::memset(hC, 0, (size_t)out_area * es);
            bp_alloc_bands(mem, mem.bp, ctx->ooc_buffers, band_bytes, nbands);
        }
        const int64_t L = std::max(Hm, Wm);
        Ap = dalloc(mem, (size_t)Hm * fb * es);
        Bp = dalloc(mem, (size_t)fb * Wm * es);
        Bt = dalloc(mem, (size_t)Wm * fb * es);
        if (dt == FPM_F32) {
            ah = dalloc(mem, (size_t)Hm * fb * op);
            al = dalloc(mem, (size_t)Hm * fb * op);
            bh = dalloc(mem, (size_t)Wm * fb * op);
            bl = dalloc(mem, (size_t)Wm * fb * op);
            sa = static_cast<float*>(dalloc(mem, (size_t)Hm * 4));
            sb = static_cast<float*>(dalloc(mem, (size_t)Wm * 4));
            bool fused = false;
            for (const Shape& x : shp)
                fused = fused || (!ooc_at(x.h * b, x.w * b) && fused_staging_applies(ctx, *d, b, x.h * b, x.w * b, true));
            if (fused) {
                ah2 = dalloc(mem, (size_t)Hm * fb * op);
                al2 = dalloc(mem, (size_t)Hm * fb * op);
                bh2 = dalloc(mem, (size_t)Wm * fb * op);
                bl2 = dalloc(mem, (size_t)Wm * fb * op);
                sa2 = static_cast<float*>(dalloc(mem, (size_t)Hm * 4));
                sb2 = static_cast<float*>(dalloc(mem, (size_t)Wm * 4));
                bmax = static_cast<unsigned*>(dalloc(mem, (size_t)Wm * sizeof(unsigned)));
                ctr = static_cast<unsigned*>(dalloc(mem, 2 * sizeof(unsigned)));
                CU(cudaMemsetAsync(bmax, 0, (size_t)Wm * sizeof(unsigned), d->s_comp));
                CU(cudaMemsetAsync(ctr, 0, 2 * sizeof(unsigned), d->s_comp));
            }
        }
        launch_fill_synthetic(Ap, dt == FPM_F64, fb, 101, L, 0, 0, Hm, fb, FPM_DIST_PM1, d->s_comp);
        launch_fill_synthetic(Bp, dt == FPM_F64, Wm, 102, L, 0, 0, fb, Wm, FPM_DIST_PM1, d->s_comp);
        if (C) CU(cudaMemsetAsync(C, 0, (size_t)in_area * es, d->s_comp));
    }
    ~GpuRunner() {
        free_problem(mem);
        bp_destroy(mem.bp);
    }

    // enqueue one run on the device's compute stream
    void run(const Shape& x) {
        const int64_t Mx = x.h * b, Nx = x.w * b;
        const cudaStream_t st = d->s_comp;
        const bool ooc = ooc_at(Mx, Nx);
        BandCall bc;
        bc.reverse = ctx->ooc_keep && (runs & 1);
        bc.kept_head = ctx->ooc_keep && runs > 0;
        bc.keep_tail = ctx->ooc_keep;
        ++runs;
        if (dt == FPM_F32) {
            // operand sets: [0] = ah / al / bh / bl / sa / sb, [1] = the *2 buffers
            void* const AH[2] = {ah, ah2};
            void* const AL[2] = {al, al2};
            void* const BH[2] = {bh, bh2};
            void* const BL[2] = {bl, bl2};
            float* const SA[2] = {sa, sa2};
            float* const SB[2] = {sb, sb2};
            const bool fused = !ooc && ah2 != nullptr && fused_staging_applies(ctx, *d, b, Mx, Nx, true);
            int s0 = fused ? cur : 0;
            StageJob job;
            if (fused) {
                if (held[s0][0] != Mx || held[s0][1] != Nx) {  // first run at this shape: stage it alone
                    launch_split_rows(static_cast<const float*>(Ap), fb, Mx, fb, sch, AH[s0], AL[s0], SA[s0], st);
                    launch_split_cols(static_cast<const float*>(Bp), Wm, fb, Nx, sch, BH[s0], BL[s0], SB[s0], st);
                }
                // the update's staging warps stage the same panels into the other set (the next run's)
                const int s1 = s0 ^ 1;
                job.nseg = 1;
                job.K = fb;
                job.lda = fb;
                job.ld_out = fb;
                job.a[0] = StagePiece{static_cast<const float*>(Ap), 0, 0, Mx};
                job.npieces = 1;
                job.b_src = static_cast<const float*>(Bp);
                job.ldb = Wm;
                job.Kb = fb;
                job.W = Nx;
                job.a_hi = AH[s1];
                job.a_lo = AL[s1];
                job.sa = SA[s1];
                job.b_hi = BH[s1];
                job.b_lo = BL[s1];
                job.sb = SB[s1];
                job.bmax = bmax;
                job.ctr = ctr;
                job.active = 1;
                held[s0][0] = held[s1][0] = Mx;
                held[s0][1] = held[s1][1] = Nx;
                cur = s1;
            } else {
                launch_split_rows(static_cast<const float*>(Ap), fb, Mx, fb, sch, ah, al, sa, st);
                launch_split_cols(static_cast<const float*>(Bp), Wm, fb, Nx, sch, bh, bl, sb, st);
                held[0][0] = held[1][0] = -1;  // set 0 now holds a shape the fused path does not track
            }
            UpdateArgs a;
            a.a_hi = AH[s0]; a.a_lo = AL[s0]; a.bt_hi = BH[s0]; a.bt_lo = BL[s0];
            a.sa = has_scales(sch) ? SA[s0] : nullptr;
            a.sb = has_scales(sch) ? SB[s0] : nullptr;
            a.stage = job;
            a.C = static_cast<float*>(C);
            a.M = Mx; a.Nc = Nx; a.K = fb; a.ldc = Nx;
            a.scheme = sch;
            a.cta_group = ctx->cta_group;
            a.num_sms = d->num_sms;
            a.raster_group = raster_group_for(ctx, *d, sch);
            a.l2_hint_b = ctx->l2_hint_b;
            a.variant = ctx->kernel_variant;
            a.chunk_k = ctx->chunk_k;
            a.raster_snake = ctx->raster_snake != 0;
            if (ooc) {
                banded_update(mem.bp, ring_at(Mx, Nx), hC, Mx, (size_t)Nx * 4, bc, st,
                              [&](int64_t r0, int64_t m, void* band) {
                                  UpdateArgs y = a;
                                  y.a_hi = static_cast<const char*>(a.a_hi) + (size_t)r0 * fb * op;
                                  y.a_lo = static_cast<const char*>(a.a_lo) + (size_t)r0 * fb * op;
                                  y.sa = a.sa ? a.sa + r0 : nullptr;
                                  y.C = static_cast<float*>(band);
                                  y.M = m;
                                  launch_update_f32(y, st);
                              });
            } else {
                launch_update_f32(a, st);
            }
        } else {  // FP64: the fused update of the k-loop (K = f b, A rows contiguous here)
            launch_transpose_f64(static_cast<const double*>(Bp), Wm, fb, Nx, static_cast<double*>(Bt), st);
            if (ooc) {
                banded_update(mem.bp, ring_at(Mx, Nx), hC, Mx, (size_t)Nx * 8, bc, st,
                              [&](int64_t r0, int64_t m, void* band) {
                                  launch_update_f64(static_cast<const double*>(Ap) + (size_t)r0 * fb, fb,
                                                    static_cast<const double*>(Bt), static_cast<double*>(band), m,
                                                    Nx, fb, Nx, true, d->num_sms, st);
                              });
            } else {
                launch_update_f64(static_cast<const double*>(Ap), fb, static_cast<const double*>(Bt),
                                  static_cast<double*>(C), Mx, Nx, fb, Nx, true, d->num_sms, st);
            }
        }
        if (ooc) bp_join(mem.bp, st);  // the update is done when C is back in host memory
    }
};

// Q8's stop rule over repetition times: (mean, 95 % half-width, converged).
struct RepStats {
    std::vector<double> ts;
    double mean = 0.0, half = 0.0;
    double rel = 0.025;  // stop when the 95 % half-width is <= rel x mean (option "sample_rel_ci")
    bool add(double t) {
        ts.push_back(t);
        const int nr = (int)ts.size();
        mean = 0.0;
        for (double v : ts) mean += v;
        mean /= nr;
        double var = 0.0;
        for (double v : ts) var += (v - mean) * (v - mean);
        var = nr > 1 ? var / (nr - 1) : 0.0;
        half = nr > 1 ? t975(nr - 1) * std::sqrt(var / nr) : 0.0;
        return nr >= 5 && half <= rel * mean;
    }
};

// Speed function of a CPU device alone, repeated under the stop rule (Q8).
void sample_cpu(pmm_ctx* ctx, Device& d, fpm_dtype dt, int64_t b, const std::vector<Shape>& shp, double* speeds,
                double* ci, int32_t* reps_out) {
    using clk = std::chrono::steady_clock;
    CpuRunner R(ctx, &d, dt, b, shp);
    for (size_t j = 0; j < shp.size(); ++j) {
        auto run = [&] {
            const auto t0 = clk::now();
            R.run(shp[j]);
            return std::chrono::duration<double>(clk::now() - t0).count();
        };
        run();
        run();  // two warm-ups
        RepStats st;
        st.rel = ctx->sample_rel_ci;
        for (int r = 0; r < 50; ++r)
            if (st.add(run())) break;
        speeds[j] = R.flops(shp[j]) / st.mean;
        if (ci) ci[j] = st.mean > 0 ? st.half / st.mean : 0.0;
        if (reps_out) reps_out[j] = (int32_t)st.ts.size();
    }
}

// devs[i] samples shapes[i][0 .. nshapes) (all devices at once when more than one).
void sample_gpu(pmm_ctx* ctx, const std::vector<Device*>& devs, const std::vector<std::vector<Shape>>& shapes,
                fpm_dtype dt, int64_t b, double* speeds, double* ci, int32_t* reps_out) {
    const int nsizes = (int)shapes[0].size();
    struct Scratch {
        std::unique_ptr<GpuRunner> R;
        cudaEvent_t e0 = nullptr, e1 = nullptr;
        RepStats st;
        int k = 1;            // kernel runs per timed repetition (concurrent sampling)
        double t_warm = 0.0;  // last warm-up run
        bool done = false;
        ~Scratch() {
            if (e0) cudaEventDestroy(e0);
            if (e1) cudaEventDestroy(e1);
        }
    };
    std::vector<std::unique_ptr<Scratch>> S;
    for (size_t i = 0; i < devs.size(); ++i) {
        S.emplace_back(new Scratch);
        Scratch& s = *S.back();
        s.R.reset(new GpuRunner(ctx, devs[i], dt, b, shapes[i]));
        CU(cudaEventCreate(&s.e0));
        CU(cudaEventCreate(&s.e1));
    }
    for (int j = 0; j < nsizes; ++j) {
        for (auto& sp : S) {
            sp->st = RepStats{};
            sp->st.rel = ctx->sample_rel_ci;
            sp->done = false;
            sp->R->runs = 0;
        }
        for (int w = 0; w < 2; ++w)
            for (size_t i = 0; i < S.size(); ++i) {
                Scratch& sp = *S[i];
                CU(cudaSetDevice(sp.R->d->cuda_dev));
                CU(cudaEventRecord(sp.e0, sp.R->d->s_comp));
                sp.R->run(shapes[i][j]);
                CU(cudaEventRecord(sp.e1, sp.R->d->s_comp));
            }
        // Concurrent sampling: every device must stay busy for the whole window
        // (P:10 (ii): resources "shared between the maximum number of
        // processes"), so a device that is k times faster runs its kernel k
        // times per repetition and each run is timed as the window / k.
        double t_max = 0.0;
        for (auto& sp : S) {
            CU(cudaSetDevice(sp->R->d->cuda_dev));
            CU(cudaEventSynchronize(sp->e1));
            sp->t_warm = elapsed_ms(sp->e0, sp->e1) * 1e-3;
            t_max = std::max(t_max, sp->t_warm);
        }
        for (auto& sp : S)
            sp->k = S.size() == 1 ? 1
                                  : (int)std::min<double>(64.0, std::max(1.0, std::round(t_max / std::max(sp->t_warm, 1e-9))));
        for (int r = 0; r < 50; ++r) {
            // all devices run every repetition, so contention stays the same until the last converges
            for (size_t i = 0; i < S.size(); ++i) {
                Scratch& sp = *S[i];
                CU(cudaSetDevice(sp.R->d->cuda_dev));
                CU(cudaEventRecord(sp.e0, sp.R->d->s_comp));
                for (int q = 0; q < sp.k; ++q) sp.R->run(shapes[i][j]);
                CU(cudaEventRecord(sp.e1, sp.R->d->s_comp));
            }
            bool all_done = true;
            for (auto& sp : S) {
                CU(cudaSetDevice(sp->R->d->cuda_dev));
                CU(cudaEventSynchronize(sp->e1));
                sp->done = sp->st.add(elapsed_ms(sp->e0, sp->e1) * 1e-3 / sp->k);
                all_done = all_done && sp->done;
            }
            if (all_done) break;
        }
        for (size_t i = 0; i < S.size(); ++i) {
            const Scratch& s = *S[i];
            // one timed run = f pivots of the x-block kernel: 2 x b^3 f flop
            speeds[i * nsizes + j] = s.R->flops(shapes[i][j]) / s.st.mean;
            if (ci) ci[i * nsizes + j] = s.st.mean > 0 ? s.st.half / s.st.mean : 0.0;
            if (reps_out) reps_out[i * nsizes + j] = (int32_t)s.st.ts.size();
        }
    }
}

// Synchronised sampling of a context with CPU devices (dev = -1; P:10 (ii)):
// every device -- GPU or CPU -- runs on a host thread of its own, all start each
// repetition together at a barrier and keep running their kernel for the same
// wall-clock window (long enough for >= 4 runs of the slowest); a device's
// speed is its completed runs' flops over their time.  Repetitions follow Q8.
void sample_sync(pmm_ctx* ctx, const std::vector<Device*>& devs, const std::vector<std::vector<Shape>>& shapes,
                 fpm_dtype dt, int64_t b, double* speeds, double* ci, int32_t* reps_out) {
    using clk = std::chrono::steady_clock;
    const int nsizes = (int)shapes[0].size();
    const size_t P = devs.size();
    std::vector<std::unique_ptr<GpuRunner>> G(P);
    std::vector<std::unique_ptr<CpuRunner>> Cr(P);
    for (size_t i = 0; i < P; ++i) {
        if (devs[i]->cpu) Cr[i].reset(new CpuRunner(ctx, devs[i], dt, b, shapes[i]));
        else G[i].reset(new GpuRunner(ctx, devs[i], dt, b, shapes[i]));
    }
    for (size_t i = 0; i < P; ++i)
        if (G[i]) {
            CU(cudaSetDevice(devs[i]->cuda_dev));
            CU(cudaStreamSynchronize(devs[i]->s_comp));
        }
    // one run, completed on return (GPU: enqueue and wait for its stream)
    auto run_once = [&](size_t i, const Shape& x) {
        if (Cr[i]) {
            Cr[i]->run(x);
        } else {
            CU(cudaSetDevice(devs[i]->cuda_dev));
            G[i]->run(x);
            CU(cudaStreamSynchronize(devs[i]->s_comp));
        }
    };
    auto flops = [&](size_t i, const Shape& x) { return Cr[i] ? Cr[i]->flops(x) : G[i]->flops(x); };
    for (int j = 0; j < nsizes; ++j) {
        std::vector<RepStats> st(P);
        for (auto& x : st) x.rel = ctx->sample_rel_ci;
        std::vector<double> t_run(P, 0.0), rate(P, 0.0);
        std::vector<std::exception_ptr> errs(P);
        double window = 0.0;
        for (size_t i = 0; i < P; ++i)
            if (G[i]) G[i]->runs = 0;
        // phase 0: warm-ups (each device alone, then the window from the slowest)
        for (size_t i = 0; i < P; ++i) {
            run_once(i, shapes[i][j]);
            const auto t0 = clk::now();
            run_once(i, shapes[i][j]);
            t_run[i] = std::chrono::duration<double>(clk::now() - t0).count();
            window = std::max(window, 4.0 * t_run[i]);
        }
        window = std::max(window, 0.02);
        bool stop = false;
        std::mutex mu;
        std::condition_variable cv;
        int arrived = 0;
        uint64_t gen = 0;
        auto barrier = [&] {
            std::unique_lock<std::mutex> lk(mu);
            const uint64_t g = gen;
            if (++arrived == (int)P) {
                arrived = 0;
                ++gen;
                cv.notify_all();
            } else {
                cv.wait(lk, [&] { return gen != g; });
            }
        };
        std::vector<std::thread> th;
        std::vector<char> failed(P, 0);
        for (size_t i = 0; i < P; ++i)
            th.emplace_back([&, i] {
                // a failing device keeps arriving at the barriers (nobody waits forever)
                for (int r = 0; r < 50; ++r) {
                    barrier();                               // everyone starts the window together
                    if (!failed[i]) {
                        try {
                            const auto t0 = clk::now();
                            int runs = 0;
                            double t_done = 0.0;
                            do {
                                run_once(i, shapes[i][j]);
                                ++runs;
                                t_done = std::chrono::duration<double>(clk::now() - t0).count();
                            } while (t_done < window);
                            rate[i] = (double)runs / t_done;  // runs per second
                        } catch (...) {
                            errs[i] = std::current_exception();
                            failed[i] = 1;
                        }
                    }
                    barrier();                               // window over for everyone
                    if (i == 0) {
                        bool all = true, bad = false;
                        for (size_t q = 0; q < P; ++q) {
                            bad = bad || failed[q];
                            if (!failed[q]) all = st[q].add(1.0 / rate[q]) && all;
                        }
                        stop = all || bad;
                    }
                    barrier();
                    if (stop) break;
                }
            });
        for (auto& t : th) t.join();
        for (auto& e : errs)
            if (e) std::rethrow_exception(e);
        for (size_t i = 0; i < P; ++i) {
            speeds[i * nsizes + j] = flops(i, shapes[i][j]) / st[i].mean;
            if (ci) ci[i * nsizes + j] = st[i].mean > 0 ? st[i].half / st[i].mean : 0.0;
            if (reps_out) reps_out[i * nsizes + j] = (int32_t)st[i].ts.size();
        }
    }
}

// fpm_sample / fpm_sample_rects: shapes per device (dev = -1: every device of
// the context at once, shapes device-major, p x nshapes).
void sample_shapes(pmm_ctx* ctx, int dev, fpm_dtype dt, int64_t b, const std::vector<std::vector<Shape>>& shapes,
                   double* speeds, double* ci, int32_t* reps_out) {
    FPM_CHECK_ARG(dt == FPM_F32 || dt == FPM_F64, "unknown dtype");
    FPM_CHECK_ARG(dt == FPM_F64 ? b % 8 == 0 && b >= 8 : b % 32 == 0 && b >= 32, "bad block size b");
    FPM_CHECK_ARG(!shapes.empty() && !shapes[0].empty() && speeds, "bad sizes");
    for (const auto& v : shapes)
        for (const Shape& x : v) FPM_CHECK_ARG(x.h >= 1 && x.w >= 1, "shape %lld x %lld", (long long)x.h, (long long)x.w);
    std::vector<Device*> devs;
    if (dev == -1) {
        for (auto& d : ctx->devs) devs.push_back(&d);
        if (has_cpu(ctx)) {  // host threads for every device, windows in step (P:10 (ii))
            FPM_CHECK_ARG(shapes.size() == devs.size(), "expected shapes for %zu devices", devs.size());
            return sample_sync(ctx, devs, shapes, dt, b, speeds, ci, reps_out);
        }
    } else {
        Device* d = local_dev(ctx, dev);
        FPM_CHECK_ARG(d != nullptr, "device %d is not driven by this context", dev);
        if (d->cpu) return sample_cpu(ctx, *d, dt, b, shapes[0], speeds, ci, reps_out);
        devs.push_back(d);
    }
    FPM_CHECK_ARG(shapes.size() == devs.size(), "expected shapes for %zu devices", devs.size());
    sample_gpu(ctx, devs, shapes, dt, b, speeds, ci, reps_out);
}

void sample(pmm_ctx* ctx, int dev, fpm_dtype dt, int64_t b, const int64_t* sizes, int nsizes, double* speeds,
            double* ci, int32_t* reps_out) {
    FPM_CHECK_ARG(nsizes >= 1 && sizes && speeds, "bad sizes");
    const std::vector<int64_t> ms = sample_sides(sizes, nsizes);
    std::vector<Shape> sq;
    for (int64_t m : ms) sq.push_back({m, m});
    const size_t ndev = dev == -1 ? ctx->devs.size() : 1;
    sample_shapes(ctx, dev, dt, b, std::vector<std::vector<Shape>>(ndev, sq), speeds, ci, reps_out);
}

}  // namespace
}  // namespace fpm

// =================================================================== C ABI
using fpm::guarded;

extern "C" int pmm_create_local(int32_t p, const int32_t* cuda_devices, const int32_t* sm_caps, pmm_ctx** out) {
    return guarded([&] {
        FPM_CHECK_ARG(out != nullptr, "null out");
        *out = nullptr;
        FPM_CHECK_ARG(p >= 1 && p <= FPM_MAX_DEVICES, "p = %d out of [1, %d]", p, FPM_MAX_DEVICES);
        FPM_CHECK_ARG(cuda_devices != nullptr, "null cuda_devices");
        bool any_gpu = false;
        for (int i = 0; i < p; ++i) {
            FPM_CHECK_ARG(cuda_devices[i] >= 0 || cuda_devices[i] == FPM_CPU_DEVICE, "bad device %d",
                          cuda_devices[i]);
            any_gpu = any_gpu || cuda_devices[i] >= 0;
        }
        int count = 0;
        if (any_gpu) CU(cudaGetDeviceCount(&count));
        // CPU devices: consecutive cores of the affinity mask; with GPUs in the
        // context the first core stays with the thread that drives them ("a
        // CPU core is usually dedicated to deal with the GPU")
        const int ncores = (int)fpm::cpu::allowed_cores().size();
        int next_core = any_gpu ? 1 : 0;
        auto ctx = std::make_unique<pmm_ctx>();
        ctx->devs.resize(p);
        try {
            for (int i = 0; i < p; ++i) {
                ctx->devs[i].idx = i;
                if (cuda_devices[i] == FPM_CPU_DEVICE) {
                    fpm::Device& d = ctx->devs[i];
                    d.cpu = true;
                    d.cuda_dev = -1;
                    d.cores = (sm_caps && sm_caps[i] > 0) ? sm_caps[i] : ncores - next_core;
                    d.first_core = next_core;
                    if (d.cores < 1 || next_core + d.cores > ncores)
                        fpm::fail(FPM_EUNSUPPORTED, "CPU device %d: %d cores requested, %d of %d left", i, d.cores,
                                  ncores - next_core, ncores);
                    next_core += d.cores;
                    fpm::init_device(d);
                    continue;
                }
                FPM_CHECK_ARG(cuda_devices[i] < count, "CUDA device %d out of range", cuda_devices[i]);
                ctx->devs[i].cuda_dev = cuda_devices[i];
                ctx->devs[i].sm_cap = sm_caps ? sm_caps[i] : 0;
                fpm::init_device(ctx->devs[i]);
            }
            // peer access between distinct GPUs (pivot copies over NVLink)
            for (int i = 0; i < p; ++i)
                for (int j = 0; j < p; ++j) {
                    const int a = cuda_devices[i], c = cuda_devices[j];
                    if (a == c || a < 0 || c < 0) continue;
                    int can = 0;
                    cudaDeviceCanAccessPeer(&can, a, c);
                    if (can) {
                        cudaSetDevice(a);
                        cudaDeviceEnablePeerAccess(c, 0);
                        cudaGetLastError();  // already enabled is fine
                    }
                }
        } catch (...) {
            for (auto& d : ctx->devs) fpm::destroy_device(d);
            throw;
        }
        *out = ctx.release();
    });
}

extern "C" int pmm_nccl_unique_id(uint8_t id_out[128]) {
    return guarded([&] {
        FPM_CHECK_ARG(id_out != nullptr, "null id");
        ncclUniqueId id;
        NC(fpm::nccl().GetUniqueId(&id));
        static_assert(sizeof(id) == 128, "ncclUniqueId size");
        std::memcpy(id_out, &id, 128);
    });
}

extern "C" int pmm_create_nccl(int32_t rank, int32_t world, int32_t cuda_device, int32_t sm_cap,
                               const uint8_t nccl_id[128], pmm_ctx** out) {
    return guarded([&] {
        FPM_CHECK_ARG(out != nullptr && nccl_id != nullptr, "null argument");
        *out = nullptr;
        FPM_CHECK_ARG(world >= 1 && world <= FPM_MAX_DEVICES && rank >= 0 && rank < world, "bad rank/world");
        int count = 0;
        CU(cudaGetDeviceCount(&count));
        FPM_CHECK_ARG(cuda_device >= 0 && cuda_device < count, "CUDA device %d out of range", cuda_device);
        auto ctx = std::make_unique<pmm_ctx>();
        ctx->nccl_mode = true;
        ctx->rank = rank;
        ctx->world = world;
        ctx->devs.resize(1);
        ctx->devs[0].idx = rank;
        ctx->devs[0].cuda_dev = cuda_device;
        ctx->devs[0].sm_cap = sm_cap;
        fpm::init_device(ctx->devs[0]);
        ncclUniqueId id;
        std::memcpy(&id, nccl_id, 128);
        CU(cudaSetDevice(cuda_device));
        ncclConfig_t cfg = fpm::nccl_config();
        ncclResult_t r = fpm::nccl().CommInitRankConfig(&ctx->world_comm, world, id, rank, &cfg);
        if (r != ncclSuccess) {
            fpm::destroy_device(ctx->devs[0]);
            fpm::fail(FPM_ENCCL, "ncclCommInitRankConfig: %s", fpm::nccl().GetErrorString(r));
        }
        int cn = 0;
        if (fpm::nccl().CommCount(ctx->world_comm, &cn) != ncclSuccess || cn != world) {
            fpm::nccl().CommDestroy(ctx->world_comm);
            fpm::destroy_device(ctx->devs[0]);
            fpm::fail(FPM_ENCCL, "world communicator has %d ranks, expected %d", cn, world);
        }
        *out = ctx.release();
    });
}

extern "C" int pmm_create_ipc(int32_t rank, int32_t world, int32_t cuda_device, int32_t sm_cap, pmm_ctx** out) {
    return guarded([&] {
        FPM_CHECK_ARG(out != nullptr, "null argument");
        *out = nullptr;
        FPM_CHECK_ARG(world >= 1 && world <= FPM_MAX_DEVICES && rank >= 0 && rank < world, "bad rank/world");
        int count = 0;
        CU(cudaGetDeviceCount(&count));
        FPM_CHECK_ARG(cuda_device >= 0 && cuda_device < count, "CUDA device %d out of range", cuda_device);
        auto ctx = std::make_unique<pmm_ctx>();
        ctx->ipc_mode = true;
        ctx->rank = rank;
        ctx->world = world;
        ctx->peer_A.assign(world, nullptr);
        ctx->peer_B.assign(world, nullptr);
        ctx->peer_flag.assign(world, nullptr);
        ctx->devs.resize(1);
        ctx->devs[0].idx = rank;
        ctx->devs[0].cuda_dev = cuda_device;
        ctx->devs[0].sm_cap = sm_cap;
        fpm::init_device(ctx->devs[0]);
        *out = ctx.release();
    });
}

namespace {
constexpr uint32_t kIpcMagic = 0x46504d31;  // "FPM1"
struct IpcBlob {
    uint32_t magic;
    int32_t rank;
    int32_t live;
    int32_t pad;
    int64_t N, b;
    cudaIpcMemHandle_t A, B;
};
static_assert(sizeof(IpcBlob) <= FPM_IPC_BLOB_BYTES, "IPC blob size");
}  // namespace

extern "C" int pmm_ipc_export(pmm_ctx* ctx, uint8_t blob_out[FPM_IPC_BLOB_BYTES]) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx && blob_out, "null argument");
        FPM_CHECK_ARG(ctx->ipc_mode, "not an IPC context");
        if (!ctx->have_problem) fpm::fail(FPM_ESTATE, "pmm_ipc_export before pmm_setup");
        IpcBlob blob;
        std::memset(&blob, 0, sizeof(blob));
        blob.magic = kIpcMagic;
        blob.rank = ctx->rank;
        blob.N = ctx->N;
        blob.b = ctx->b;
        fpm::Device& d = ctx->devs[0];
        blob.live = d.live() ? 1 : 0;
        if (d.live()) {
            CU(cudaSetDevice(d.cuda_dev));
            CU(cudaIpcGetMemHandle(&blob.A, d.A));
            CU(cudaIpcGetMemHandle(&blob.B, d.B));
        }
        std::memset(blob_out, 0, FPM_IPC_BLOB_BYTES);
        std::memcpy(blob_out, &blob, sizeof(blob));
    });
}

extern "C" int pmm_ipc_import(pmm_ctx* ctx, const uint8_t* blobs, int32_t world) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx && blobs, "null argument");
        FPM_CHECK_ARG(ctx->ipc_mode, "not an IPC context");
        FPM_CHECK_ARG(world == ctx->world, "expected %d blobs", ctx->world);
        if (!ctx->have_problem) fpm::fail(FPM_ESTATE, "pmm_ipc_import before pmm_setup");
        fpm::close_peers(ctx);
        fpm::drop_graph(ctx);
        CU(cudaSetDevice(ctx->devs[0].cuda_dev));
        for (int q = 0; q < world; ++q) {
            IpcBlob blob;
            std::memcpy(&blob, blobs + (size_t)q * FPM_IPC_BLOB_BYTES, sizeof(blob));
            FPM_CHECK_ARG(blob.magic == kIpcMagic && blob.rank == q, "blob %d is not rank %d's export", q, q);
            FPM_CHECK_ARG(blob.N == ctx->N && blob.b == ctx->b, "rank %d set up a different problem", q);
            const colpart_rect& r = ctx->rects[q];
            FPM_CHECK_ARG((blob.live != 0) == (r.h > 0 && r.w > 0), "rank %d liveness differs from the arrangement", q);
            if (q == ctx->rank || !blob.live) continue;
            CU(cudaIpcOpenMemHandle(&ctx->peer_A[q], blob.A, cudaIpcMemLazyEnablePeerAccess));
            CU(cudaIpcOpenMemHandle(&ctx->peer_B[q], blob.B, cudaIpcMemLazyEnablePeerAccess));
            const size_t qHW = (size_t)(r.h * ctx->b) * (size_t)(r.w * ctx->b) * fpm::esize(ctx->dt);
            ctx->peer_flag[q] = reinterpret_cast<uint64_t*>(static_cast<char*>(ctx->peer_B[q]) + (qHW + 63) / 64 * 64);
        }
        ctx->peers_ready = true;
    });
}

extern "C" int pmm_destroy(pmm_ctx* ctx) {
    return guarded([&] {
        if (!ctx) return;
        fpm::close_peers(ctx);
        fpm::drop_graph(ctx);
        if (ctx->ev_fork) cudaEventDestroy(ctx->ev_fork);
        for (auto& d : ctx->devs) fpm::destroy_device(d);
        if (ctx->nccl_mode) {
            if (ctx->col_comm) fpm::nccl().CommDestroy(ctx->col_comm);
            if (ctx->world_comm) fpm::nccl().CommDestroy(ctx->world_comm);
        }
        delete ctx;
    });
}

extern "C" int pmm_set_option(pmm_ctx* ctx, const char* key, int64_t value) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx && key, "null argument");
        fpm::drop_graph(ctx);  // every option can change the captured k-loop
        const std::string k(key);
        if (k == "graph") {
            FPM_CHECK_ARG(value == 0 || value == 1, "graph must be 0 or 1");
            ctx->graph = (int)value;
        } else if (k == "f32_scheme") {
            FPM_CHECK_ARG(value == -1 || value == 0 || value == 1 || value == 3,
                          "f32_scheme must be -1 (auto), 0 (F16X3), 1 (TF32X3) or 3 (F16I8)");
            if (ctx->f32_scheme != (int)value) ctx->have_problem = false;  // operand buffers change size
            ctx->f32_scheme = (int)value;
        } else if (k == "cta_group") {
            FPM_CHECK_ARG(value == 1 || value == 2, "cta_group must be 1 or 2");
            ctx->cta_group = (int)value;
        } else if (k == "fuse") {
            FPM_CHECK_ARG(value >= 0 && value <= 8, "fuse must be 0 (auto) or 1..8");
            if (ctx->fuse != (int)value) ctx->have_problem = false;  // staging buffers change size
            ctx->fuse = (int)value;
        } else if (k == "tail_stream") {
            FPM_CHECK_ARG(value == 0 || value == 1, "tail_stream must be 0 or 1");
            ctx->tail_stream = (int)value;
        } else if (k == "e2e_tail") {
            FPM_CHECK_ARG(value >= -1 && value <= fpm::kMaxTail, "e2e_tail must be -1 (auto), 0 (off) or 1..%d",
                          fpm::kMaxTail);
            ctx->e2e_tail = (int)value;
        } else if (k == "tail_fuse") {
            FPM_CHECK_ARG(value == 0 || value == 1, "tail_fuse must be 0 or 1");
            ctx->tail_fuse = (int)value;
        } else if (k == "tail_band") {
            FPM_CHECK_ARG(value >= 256 && value % 256 == 0, "tail_band must be a positive multiple of 256 rows");
            ctx->tail_band = value;
        } else if (k == "sm_partition") {
            FPM_CHECK_ARG(value == 0 || value == 1, "sm_partition must be 0 (grid caps) or 1 (green contexts)");
            if (ctx->sm_partition != (int)value) {
                fpm::set_sm_partition(ctx, value == 1);
                ctx->sm_partition = (int)value;
            }
        } else if (k == "ooc_buffers") {
            FPM_CHECK_ARG(value >= 2 && value <= fpm::kMaxBandBufs, "ooc_buffers must be in [2, %d]",
                          fpm::kMaxBandBufs);
            if (ctx->ooc_buffers != (int)value) ctx->have_problem = false;  // band buffers change
            ctx->ooc_buffers = (int)value;
        } else if (k == "ooc_keep") {
            FPM_CHECK_ARG(value == 0 || value == 1, "ooc_keep must be 0 or 1");
            ctx->ooc_keep = (int)value;
        } else if (k == "kernel_variant") {
            FPM_CHECK_ARG((value >= -1 && value <= 8) || value == 12 || value == 13,
                          "kernel_variant must be -1 (auto), 0..8 (6: F16I8 only; 7, 8: F16X3 / TF32X3 only) "
                          "or 12, 13 (F16X3 on clusters of two CTA pairs, B multicast)");
            ctx->kernel_variant = (int)value;
        } else if (k == "share_b") {
            FPM_CHECK_ARG(value == 0 || value == 1, "share_b must be 0 or 1");
            ctx->share_b = (int)value;
        } else if (k == "fused_staging") {
            FPM_CHECK_ARG(value >= 0 && value <= 2, "fused_staging must be 0, 1 (where it pays) or 2 (always)");
            ctx->fused_staging = (int)value;
        } else if (k == "sample_rel_ci_permille") {
            FPM_CHECK_ARG(value >= 1 && value <= 500, "sample_rel_ci_permille must be in [1, 500]");
            ctx->sample_rel_ci = value / 1000.0;
        } else if (k == "raster_snake") {
            FPM_CHECK_ARG(value == 0 || value == 1, "raster_snake must be 0 or 1");
            ctx->raster_snake = (int)value;
        } else if (k == "chunk_k") {
            FPM_CHECK_ARG(value >= 0 && value <= (1 << 20), "chunk_k must be 0 (auto = 512) or a positive K");
            ctx->chunk_k = (int)value;
        } else if (k == "l2_hint_b") {
            FPM_CHECK_ARG(value >= 0 && value <= 2, "l2_hint_b must be 0 (normal), 1 (first) or 2 (last)");
            ctx->l2_hint_b = (int)value;
        } else if (k == "raster_group") {
            FPM_CHECK_ARG(value >= 0 && value <= 4096, "raster_group must be 0 (auto) or in [1, 4096]");
            ctx->raster_group = (int)value;
        } else {
            fpm::fail(FPM_EINVAL, "unknown option '%s'", key);
        }
    });
}

extern "C" int pmm_set_device_option(pmm_ctx* ctx, int32_t dev, const char* key, int64_t value) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx && key, "null argument");
        fpm::Device* d = fpm::local_dev(ctx, dev);
        FPM_CHECK_ARG(d != nullptr, "device %d is not driven by this context", dev);
        fpm::drop_graph(ctx);
        const std::string k(key);
        if (k == "cpu_first_core") {  // CPU device: move its team to cores [value, value + c) of the affinity mask
            FPM_CHECK_ARG(d->cpu, "cpu_first_core applies to CPU devices only");
            FPM_CHECK_ARG(value >= 0, "cpu_first_core must be >= 0");
            if (d->first_core != (int)value) {
                const int old = d->first_core;
                fpm::cpu::team_destroy(d->team);
                d->team = nullptr;
                d->first_core = (int)value;
                try {
                    fpm::init_device(*d);
                } catch (...) {
                    d->first_core = old;
                    fpm::init_device(*d);
                    throw;
                }
            }
        } else if (k == "c_cap_bytes") {
            FPM_CHECK_ARG(!d->cpu, "c_cap_bytes applies to GPU devices");
            FPM_CHECK_ARG(value >= 0, "c_cap_bytes must be >= 0");
            if (d->c_cap != value) ctx->have_problem = false;  // C_i placement changes
            d->c_cap = value;
        } else {
            fpm::fail(FPM_EINVAL, "unknown device option '%s'", key);
        }
    });
}

extern "C" int pmm_setup(pmm_ctx* ctx, int64_t N, int64_t b, int32_t p, const colpart_rect* rects, fpm_dtype dt) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr, "null ctx");
        fpm::setup(ctx, N, b, p, rects, dt);
    });
}

extern "C" int pmm_upload(pmm_ctx* ctx, const void* A, const void* B, int64_t ld, int64_t row_base,
                          int64_t col_base) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr, "null ctx");
        fpm::upload(ctx, A, B, ld, row_base, col_base, nullptr);
    });
}

extern "C" int pmm_fill_synthetic(pmm_ctx* ctx, uint64_t seed_a, uint64_t seed_b, int32_t dist) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr, "null ctx");
        fpm::fill_synthetic(ctx, seed_a, seed_b, dist);
    });
}

extern "C" int pmm_compute(pmm_ctx* ctx, int32_t zero_c, pmm_stats* stats) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr, "null ctx");
        (void)zero_c;  // every compute produces C = A B (iteration 0 overwrites C)
        fpm::compute(ctx, stats);
    });
}

extern "C" int pmm_compute_into(pmm_ctx* ctx, void* C, int64_t ld, int64_t row_base, int64_t col_base,
                                pmm_stats* stats) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr && C != nullptr, "null argument");
        if (!ctx->have_problem) fpm::fail(FPM_ESTATE, "pmm_compute_into before pmm_setup");
        for (auto& d : ctx->devs)
            if (d.live()) fpm::check_window(ctx, d, ld, row_base, col_base);
        const fpm::HostDst out{C, ld, row_base, col_base};
        pmm_stats local;
        std::vector<char> done;
        fpm::compute(ctx, &local, nullptr, &out, &done);
        double td = 0.0;
        fpm::download(ctx, C, ld, row_base, col_base, &td, &done);
        local.t_download_s = std::max(local.t_download_s, td);
        if (stats) *stats = local;
    });
}

extern "C" int pmm_download(pmm_ctx* ctx, void* C, int64_t ld, int64_t row_base, int64_t col_base) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr, "null ctx");
        fpm::download(ctx, C, ld, row_base, col_base, nullptr);
    });
}

extern "C" int pmm_download_block(pmm_ctx* ctx, int64_t r0, int64_t c0, int64_t rows, int64_t cols, void* C_host,
                                  int64_t ld) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr && C_host != nullptr, "null argument");
        if (!ctx->have_problem) fpm::fail(FPM_ESTATE, "pmm_download_block before pmm_setup");
        FPM_CHECK_ARG(rows >= 0 && cols >= 0 && ld >= cols, "bad block shape");
        if (rows == 0 || cols == 0) return;
        const int64_t b = ctx->b;
        const size_t es = ctx->dt == FPM_F64 ? 8 : 4;
        for (auto& d : ctx->devs) {
            if (!d.live()) continue;
            const int64_t R0 = d.rect.row0 * b, C0 = d.rect.col0 * b;
            if (r0 >= R0 && c0 >= C0 && r0 + rows <= R0 + d.H && c0 + cols <= C0 + d.W) {
                const size_t off0 = ((size_t)(r0 - R0) * d.W + (size_t)(c0 - C0)) * es;
                if (d.cpu) {
                    fpm::copy_rows(C_host, ld * es, static_cast<const char*>(d.C) + off0, d.W * es, cols * es, rows);
                    return;
                }
                CU(cudaSetDevice(d.cuda_dev));
                CU(cudaStreamSynchronize(d.s_comp));
                const size_t off = ((size_t)(r0 - R0) * d.W + (size_t)(c0 - C0)) * es;
                if (d.ooc) {
                    CU(cudaStreamSynchronize(d.bp.s_d2h));
                    fpm::copy_rows(C_host, ld * es, reinterpret_cast<const char*>(d.hC) + off, d.W * es, cols * es,
                                   rows);
                } else {
                    CU(cudaMemcpy2D(C_host, ld * es, static_cast<const char*>(d.C) + off, d.W * es, cols * es, rows,
                                    cudaMemcpyDeviceToHost));
                }
                return;
            }
        }
        fpm::fail(FPM_EINVAL, "block not inside one local rectangle");
    });
}

extern "C" int pmm_group_times(pmm_ctx* ctx, int32_t dev, double* out, int32_t cap, int32_t* count) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr && count != nullptr && (cap == 0 || out != nullptr), "null argument");
        if (!ctx->have_problem) fpm::fail(FPM_ESTATE, "pmm_group_times before pmm_setup");
        fpm::Device* d = fpm::local_dev(ctx, dev);
        FPM_CHECK_ARG(d != nullptr, "device %d is not driven by this process", dev);
        FPM_CHECK_ARG(!d->cpu, "device %d is a host-CPU device (its times are host-timed)", dev);
        const int ng = d->live() ? (int)ctx->groups.size() : 0;
        *count = ng;
        if (ng == 0) return;
        CU(cudaSetDevice(d->cuda_dev));
        CU(cudaEventSynchronize(d->ev_stop));
        auto rel = [&](cudaEvent_t e) {  // seconds after ev_start; NaN for an event this loop did not record
            float ms = 0.0f;
            if (cudaEventElapsedTime(&ms, d->ev_start, e) != cudaSuccess) {
                cudaGetLastError();
                return std::nan("");
            }
            return (double)ms * 1e-3;
        };
        for (int g = 0; g < ng && 4 * g + 3 < cap; ++g) {
            out[4 * g + 0] = rel(d->ev_pack0[g]);
            out[4 * g + 1] = rel(d->ev_pack1[g]);
            out[4 * g + 2] = rel(d->ev_upd0[g]);
            out[4 * g + 3] = rel(d->ev_upd1[g]);
        }
    });
}

extern "C" int pmm_run(pmm_ctx* ctx, const void* A, const void* B, void* C, int64_t N, int64_t b, int32_t p,
                       const colpart_rect* rects, fpm_dtype dt, int64_t ld, int64_t row_base, int64_t col_base,
                       pmm_stats* stats) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr, "null ctx");
        bool same = ctx->have_problem && ctx->N == N && ctx->b == b && ctx->p == p && ctx->dt == dt;
        if (same)
            for (int i = 0; i < p; ++i) {
                const colpart_rect &x = ctx->rects[i], &y = rects[i];
                same = same && x.col == y.col && x.row0 == y.row0 && x.col0 == y.col0 && x.h == y.h && x.w == y.w;
            }
        if (ctx->ipc_mode && !(same && ctx->peers_ready))
            fpm::fail(FPM_EUNSUPPORTED, "pmm_run on an IPC context needs the same problem set up and the peers "
                                        "imported first (pmm_setup, pmm_ipc_export / import on every rank)");
        if (!same) fpm::setup(ctx, N, b, p, rects, dt);
        FPM_CHECK_ARG(A && B && C, "null host matrix");
        for (auto& d : ctx->devs)
            if (d.live()) fpm::check_window(ctx, d, ld, row_base, col_base);
        const fpm::HostSrc host{A, B, ld, row_base, col_base};
        const fpm::HostDst out{C, ld, row_base, col_base};
        pmm_stats local;
        std::vector<char> done;
        if (fpm::has_cpu(ctx)) {
            // CPU devices pull pivots from resident rectangles: every device's
            // inputs are in place before the k-loop (C still streamed out)
            double tu = 0.0;
            fpm::upload(ctx, A, B, ld, row_base, col_base, &tu);
            fpm::compute(ctx, &local, nullptr, &out, &done);
            local.t_upload_s = tu;
        } else {
            fpm::compute(ctx, &local, &host, &out, &done);  // host panels streamed in, C streamed out
        }
        double td = 0.0;
        fpm::download(ctx, C, ld, row_base, col_base, &td, &done);  // devices without a tail
        local.t_download_s = std::max(local.t_download_s, td);
        if (stats) *stats = local;
    });
}

extern "C" int fpm_sample(pmm_ctx* ctx, int32_t dev, fpm_dtype dt, int64_t b, const int64_t* sizes,
                          int32_t nsizes, double* speeds_out, double* rel_ci95_out, int32_t* reps_out) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr, "null ctx");
        fpm::sample(ctx, dev, dt, b, sizes, nsizes, speeds_out, rel_ci95_out, reps_out);
    });
}

extern "C" int fpm_sample_rects(pmm_ctx* ctx, int32_t dev, fpm_dtype dt, int64_t b, const int64_t* shapes,
                                int32_t nshapes, double* speeds_out, double* rel_ci95_out, int32_t* reps_out) {
    return guarded([&] {
        FPM_CHECK_ARG(ctx != nullptr && shapes != nullptr, "null argument");
        FPM_CHECK_ARG(nshapes >= 1, "nshapes must be >= 1");
        const size_t ndev = dev == -1 ? ctx->devs.size() : 1;
        std::vector<std::vector<fpm::Shape>> shp(ndev);
        for (size_t i = 0; i < ndev; ++i)
            for (int j = 0; j < nshapes; ++j)
                shp[i].push_back({shapes[(i * nshapes + j) * 2], shapes[(i * nshapes + j) * 2 + 1]});
        fpm::sample_shapes(ctx, dev, dt, b, shp, speeds_out, rel_ci95_out, reps_out);
    });
}

// ------------------------------------------------------- kernel-level ABI
extern "C" int fpm_k_split_f32(const float* src, int64_t ld, int64_t rows, int64_t K, int32_t scheme, void* hi,
                               void* lo, float* inv_scale, void* stream) {
    return guarded([&] {
        FPM_CHECK_ARG(scheme == 0 || scheme == 1 || scheme == 3, "scheme must be 0, 1 or 3");
        FPM_CHECK_ARG(scheme == 1 || inv_scale != nullptr, "F16X3 / F16I8 need inv_scale");
        fpm::launch_split_rows(src, ld, rows, K, (fpm::SplitScheme)scheme, hi, lo, inv_scale,
                               static_cast<cudaStream_t>(stream));
    });
}

extern "C" int fpm_k_split_cols_f32(const float* src, int64_t ld, int64_t K, int64_t W, int32_t scheme, void* hi,
                                    void* lo, float* inv_scale, void* stream) {
    return guarded([&] {
        FPM_CHECK_ARG(scheme == 0 || scheme == 1 || scheme == 3, "scheme must be 0, 1 or 3");
        fpm::launch_split_cols(src, ld, K, W, (fpm::SplitScheme)scheme, hi, lo, inv_scale,
                               static_cast<cudaStream_t>(stream));
    });
}

extern "C" int fpm_k_transpose(const void* src, int32_t dt, int64_t ld, int64_t rows, int64_t cols, void* dst,
                               void* stream) {
    return guarded([&] {
        FPM_CHECK_ARG(dt == FPM_F32 || dt == FPM_F64, "bad dtype");
        if (dt == FPM_F32)
            fpm::launch_transpose_f32(static_cast<const float*>(src), ld, rows, cols, static_cast<float*>(dst),
                                      static_cast<cudaStream_t>(stream));
        else
            fpm::launch_transpose_f64(static_cast<const double*>(src), ld, rows, cols, static_cast<double*>(dst),
                                      static_cast<cudaStream_t>(stream));
    });
}

extern "C" int fpm_k_update_f32(const void* a_hi, const void* a_lo, const void* bt_hi, const void* bt_lo,
                                const float* sa, const float* sb, float* C, int64_t M, int64_t Nc, int64_t K,
                                int64_t ldc, int32_t scheme, int32_t cta_group, int32_t num_sms, int32_t accumulate,
                                int32_t variant, void* stream) {
    return guarded([&] {
        FPM_CHECK_ARG(scheme >= 0 && scheme <= 3, "scheme must be 0, 1, 2 (int8 timing probe) or 3");
        FPM_CHECK_ARG(cta_group == 1 || cta_group == 2, "cta_group must be 1 or 2");
        FPM_CHECK_ARG((variant >= -1 && variant <= 5) || ((variant == 7 || variant == 8) && scheme != 3) ||
                          ((variant == 12 || variant == 13) && scheme == 0) ||
                          (variant >= 6 && variant <= 11 && variant != 7 && variant != 8 && scheme == 3),
                      "variant must be -1 (auto), 0..5, 7, 8, 12, 13 (F16X3), or 6, 9..11 with F16I8");
        FPM_CHECK_ARG(scheme == 1 || scheme == 2 || (sa && sb), "F16X3 / F16I8 need sa and sb");
        fpm::UpdateArgs a;
        a.a_hi = a_hi; a.a_lo = a_lo; a.bt_hi = bt_hi; a.bt_lo = bt_lo;
        a.sa = (scheme == 0 || scheme == 3) ? sa : nullptr;
        a.sb = (scheme == 0 || scheme == 3) ? sb : nullptr;
        a.C = C; a.M = M; a.Nc = Nc; a.K = K; a.ldc = ldc;
        a.scheme = (fpm::SplitScheme)scheme;
        a.cta_group = cta_group;
        int dev = 0, sms = 0;
        CU(cudaGetDevice(&dev));
        CU(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
        a.num_sms = (num_sms > 0 && num_sms < sms) ? num_sms : sms;
        a.accumulate = accumulate != 0;
        a.variant = variant;
        fpm::launch_update_f32(a, static_cast<cudaStream_t>(stream));
    });
}

extern "C" int fpm_k_prof(int32_t op, uint64_t* out) {
    return guarded([&] {
        FPM_CHECK_ARG(op >= 0 && op <= 2, "op must be 0, 1 or 2");
        FPM_CHECK_ARG(op != 2 || out != nullptr, "null out");
        fpm::update_prof(op, reinterpret_cast<unsigned long long*>(out));
    });
}

extern "C" int fpm_k_update_f64(const double* A, int64_t lda, const double* Bt, double* C, int64_t M, int64_t Nc,
                                int64_t K, int64_t ldc, int32_t accumulate, void* stream) {
    return guarded([&] {
        fpm::launch_update_f64(A, lda, Bt, C, M, Nc, K, ldc, accumulate != 0, 0, static_cast<cudaStream_t>(stream));
    });
}

extern "C" int fpm_k_fill_synthetic(void* dst, int32_t dt, int64_t ld, uint64_t seed, int64_t N, int64_t r0,
                                    int64_t c0, int64_t rows, int64_t cols, int32_t dist, void* stream) {
    return guarded([&] {
        FPM_CHECK_ARG(dt == FPM_F32 || dt == FPM_F64, "bad dtype");
        fpm::launch_fill_synthetic(dst, dt == FPM_F64, ld, seed, N, r0, c0, rows, cols, dist,
                                   static_cast<cudaStream_t>(stream));
    });
}
