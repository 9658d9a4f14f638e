// lf_internal.cuh -- internal declarations shared by liblf.so's translation
// units (never included by the oracle; never exported).
#pragma once

#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include <string>
#include <atomic>
#include <mutex>
#include <vector>

#include "liteform.h"

namespace lf {

constexpr int kMaxT = 32;  // natural buckets t = 0..31

// ceil(log2(l)) for l >= 1 (natural bucket, reading R1)
__host__ __device__ __forceinline__ int ceil_log2_i64(int64_t l) {
#ifdef __CUDA_ARCH__
    return l <= 1 ? 0 : 64 - __clzll((unsigned long long)(l - 1));
#else
    int t = 0;
    while ((int64_t(1) << t) < l) t++;
    return t;
#endif
}

// Multiprocessors of the current device (queried once per device; grids are
// sized in multiples of it, never from a hardcoded 148).
inline int sm_count() {
    static std::atomic<int> cache[64];
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) dev = 0;
    int n = cache[dev].load(std::memory_order_relaxed);
    if (n <= 0) {
        if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n <= 0) n = 1;
        cache[dev].store(n, std::memory_order_relaxed);
    }
    return n;
}
inline int current_device() {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) dev = 0;
    return dev;
}

// Per-bucket descriptor the SpMM kernel walks (device copy of the bucket
// table plus its work decomposition into warp tasks).
struct BucketDev {
    int64_t slot_off;   // first slot
    int64_t row_off;    // first CELL row
    int64_t n_slots;    // n_rows_pad * W
    int64_t task_off;   // first task index of this bucket
    int32_t t;          // log2 width
    int32_t task_slots; // slots per task: 32 (W <= 32), W (W <= 2^kPieceLog2) or 2^kPieceLog2
    int32_t piece_log2; // W >= 32: a CELL row is 2^piece_log2 tasks of <= 2^kPieceLog2 slots
    int32_t pad_;
    int64_t n_real_rows; // CELL rows before block padding
    int64_t n_rows_pad;  // CELL rows after block padding
};
// max width exponents e_p passed by value to the build kernels
struct WidthArg {
    int8_t e[LF_MAX_PARTS];
};

// Stats the configure kernels accumulate (device, zero-initialised).
struct StatsPart {
    unsigned long long H[kMaxT], F[kMaxT], Unat[kMaxT], Utop[kMaxT];
};
struct StatsDev {
    unsigned long long len_min, len_max, len_sum, len_sumsq;  // row lengths
    unsigned long long grp_union, grp_nnz;  // sampled groups of kGroupRows rows: distinct columns, nonzeros
    unsigned long long win_span, win_cnt, win_over;  // sampled groups of 128 rows: summed spans, samples, spans > 256
    StatsPart part[LF_MAX_PARTS];  // only the first P are cleared / copied back
};
inline size_t stats_bytes(int P) { return offsetof(StatsDev, part) + (size_t)P * sizeof(StatsPart); }

// ---- launchers (kernels in csrc/kernels/*.cu) ----
uint32_t mask_slots(int64_t n_cols);  // words of the column-mask array (power of two >= K)
size_t stats_scratch_bytes(int64_t n_rows, int64_t nnz, int P);  // t0 per segment + tile -> row map
cudaError_t launch_features(const lf_csr &A, StatsDev *d_stats, cudaStream_t s);  // len_* only
// sample = false: the group / window samples (independent of P) are already
// known from an earlier pass over the same A and are not recomputed
cudaError_t launch_stats(const lf_csr &A, int P, StatsDev *d_stats, uint32_t *d_colmask, uint8_t *d_t0seg,
                         cudaStream_t s, bool sample = true);

struct BuildScratch {
    int32_t *seg_rel;       // [I*(P-1)] segment starts relative to the row start (P > 1)
    long long *tile_cnt;    // [P][n_tiles][32] n_sub sums per tile -> exclusive offsets
    long long *key_total;   // [P][32]
    long long *key_row_off; // [P][32] first CELL row of bucket (p,t), -1 if none
    int64_t *src_pos;       // [R_tot] CSR position of a CELL row's first slot
    int32_t *src_cnt;       // [R_tot] real slots in the CELL row (0 for padding)
    int n_tiles;
};
constexpr int kBuildTile = 256;  // rows per tile of the bucketize passes
// A folded source row whose CELL rows all sit in one wide bucket (W >= 32)
// and number at most kMaxRun is summed by a single warp and stored once.
#ifndef LF_MAX_RUN
#define LF_MAX_RUN 8
#endif
constexpr int kMaxRun = LF_MAX_RUN;
// Work is claimed from per-launch queues in ranges of at most kWideChunk
// tasks (smaller near the end); run_bound[x] = offset (0..32) from wide task x
// to the first task that may start a claim (never inside a whole run).
#ifndef LF_WIDE_CHUNK
#define LF_WIDE_CHUNK 8
#endif
constexpr int kWideChunk = LF_WIDE_CHUNK;
// A CELL row wider than 2^kPieceLog2 slots (a large max width chosen by
// Algorithm 3, e.g. the dense rows of an arrowhead matrix) is split into
// pieces of 2^kPieceLog2 slots, separate wide tasks that red.add into the
// pre-zeroed C row, so one long row never serialises on a single warp.
#ifndef LF_PIECE_LOG2
#define LF_PIECE_LOG2 10
#endif
constexpr int kPieceLog2 = LF_PIECE_LOG2;
// CELL rows per group of the grouped SpMM path (cell_spmm.cu)
constexpr int kGroupRows = 4;
// row_mode[i]: how C row i is produced
enum : uint8_t {
    kRowPlain = 0,  // one CELL row, plain store
    kRowEmpty = 1,  // no CELL row: zeroed by the SpMM kernel's epilogue
    kRowRed = 2,    // several writers: pre-zeroed, red.global.add
    kRowRun = 3,    // a whole run (<= kMaxRun CELL rows) summed by one warp, plain store
};

cudaError_t launch_seg(const lf_csr &A, int P, int32_t *seg_rel, cudaStream_t s);
cudaError_t launch_bucket_count(const lf_csr &A, int P, const WidthArg &e, const BuildScratch &sc,
                                int32_t *row_cnt, cudaStream_t s);
// padding rows (n_real_rows .. n_rows_pad of every bucket): rowInd / tag -1,
// src_cnt 0; and the n_ctr queue counters zeroed
cudaError_t launch_pad_init(const BucketDev *bk, int nb, int32_t *row_ind, int32_t *row_tag, int32_t *src_cnt,
                            int64_t *src_pos, unsigned long long *ctr, int n_ctr, cudaStream_t s);
cudaError_t launch_tile_scan(int P, const BuildScratch &sc, cudaStream_t s);
cudaError_t launch_bucket_place(const lf_csr &A, int P, const WidthArg &e, const BuildScratch &sc,
                                const int32_t *row_cnt, int32_t *row_ind, int32_t *row_tag, uint8_t *row_mode,
                                cudaStream_t s);
cudaError_t launch_run_bounds(const BucketDev *bk_w, int nb_w, int64_t n_tasks_w, const int32_t *row_tag,
                              uint8_t *run_bound, cudaStream_t s);
cudaError_t launch_slot_fill(const lf_csr &A, const BucketDev *d_buckets, int nb, int64_t n_slots,
                             const BuildScratch &sc, int32_t *col_out, float *val_out, cudaStream_t s);

// SpMM
struct SpmmArgs {
    const BucketDev *bk_n;  // buckets with W < 32; task_off counts 32-slot tasks
    const BucketDev *bk_w;  // buckets with W >= 32; task_off counts rows
    int nb_n, nb_w;
    int64_t n_tasks_n, n_tasks_w;
    int64_t slots_n, slots_w;
    int blocks_n;  // set by the launcher
    const uint8_t *row_mode;
    int64_t n_rows;
    const uint8_t *run_bound;  // [n_tasks_w + 1]
    unsigned long long *ctr;   // [4] the handle's counter slot for this launch: wide, narrow, warps done
    const int32_t *col;
    const float *val;
    const int32_t *row_tag;
    const float *B;
    int64_t ldb;
    float *C;
    int64_t ldc;
    int J;
    // grouped path (cell_spmm.cu): every bucket W <= 32, task_off = first group
    const BucketDev *bk_g;
    int nb_g;
    int grouped;  // use it (when J and the alignment allow)
    int64_t n_groups;
    // tensor-core grouped path: the same buckets, task_off counting 16-row groups
    const BucketDev *bk_m;
    int mma;
    int64_t n_groups_m;
    // tcgen05 windowed path (cell_spmm_tc.cu): the same buckets, task_off
    // counting 128-row groups, and each group's B-row window {lo, span}
    const BucketDev *bk_t;
    int nb_t;
    int tc;
    int64_t n_groups_t;
    const int2 *tc_win;
    // fused row exchange (lf_spmm_ex): n_dst > 0 writes C row i to every
    // dst[d] + (row_base + i) * ldc instead of C (peer C buffers over NVLink)
    int n_dst;
    float *const *dst;  // (device) [n_dst]
    int64_t row_base;
    uintptr_t c_bits;   // OR of the C / destination base addresses (alignment checks)
};
constexpr int kMaxDst = 8;
// destination base d of a fused row exchange (read-only path)
__device__ __forceinline__ float *ld_dst(float *const *dst, int d) {
    return reinterpret_cast<float *>(__ldg(reinterpret_cast<const unsigned long long *>(dst) + d));
}
cudaError_t launch_cell_spmm(const SpmmArgs &a, cudaStream_t s);  // pre-zeroes kRowRed rows itself
// name of the kernel launch_cell_spmm runs for these arguments
const char *cell_spmm_path(const SpmmArgs &a);
// tcgen05 windowed path (cell_spmm_tc.cu)
constexpr int kTcGroupLog2 = 7;
constexpr int kTcGroupRows = 1 << kTcGroupLog2;
bool tc_ok(const SpmmArgs &a);
cudaError_t launch_cell_spmm_tc(const SpmmArgs &a, cudaStream_t s);
cudaError_t launch_tc_windows(const BucketDev *bk_t, int nb_t, int64_t n_groups, const int32_t *col,
                              const int32_t *src_cnt, int2 *win, cudaStream_t s);

cudaError_t launch_csr_spmm(const lf_csr &A, const float *B, int64_t ldb, int J, float *C, int64_t ldc,
                            cudaStream_t s);
cudaError_t launch_validate(const lf_csr &A, int *d_flag, cudaStream_t s);

}  // namespace lf

constexpr int kCtrSlots = 64;  // concurrent lf_spmm launches on one handle
struct lf_cell {
    lf_cell_params params;
    int64_t n_rows = 0, n_cols = 0, nnz = 0;
    int64_t n_cell_rows = 0, n_slots = 0;
    int64_t n_tasks_n = 0, n_tasks_w = 0, slots_n = 0, slots_w = 0;
    int nb_n = 0, nb_w = 0;
    int32_t *row_ind = nullptr;  // view array (bit-exact with the oracle)
    int32_t *col_ind = nullptr;
    float *val = nullptr;
    int32_t *row_tag = nullptr;  // (row << 3) | S,F,L flags (cell_spmm.cu); -1 = padding
    uint8_t *row_mode = nullptr;  // [n_rows] kRow* (how each C row is produced)
    uint8_t *run_bound = nullptr; // [n_tasks_w + 1] (in the pool)
    lf::BucketDev *d_buckets = nullptr;  // [nb] all, [nb_n] W < 32 class, [nb_w] W >= 32 class, [nb_g] grouped
    int nb_g = 0;            // grouped-path buckets (= nb when every W <= 32, else 0)
    int64_t n_groups = 0;
    int grouped = 0;         // lf_spmm takes the grouped path
    int64_t n_groups_m = 0;  // 16-row groups (tensor-core grouped path)
    int mma = 0;             // lf_spmm takes the tensor-core grouped path
    int64_t n_groups_t = 0;  // 128-row groups of the tcgen05 windowed path
    int2 *tc_win = nullptr;  // [n_groups_t] B-row window per group (in the pool; NULL: not built)
    int tc = 0;              // lf_spmm takes the tcgen05 windowed path
    // work-queue counters, kCtrSlots slots of 4 (wide, narrow, warps done, -)
    // in the pool: launch k uses slot k % kCtrSlots and its last warp resets
    // it, so lf_spmm needs no allocation or memset per call
    unsigned long long *ctr_ring = nullptr;
    mutable std::atomic<uint32_t> launch_seq{0};
    std::vector<lf_bucket> buckets;
    std::vector<lf::BucketDev> h_buckets;
    // memory: one pool allocation holds every array above
    void *pool = nullptr;
    size_t pool_bytes = 0;
    lf_allocator al{};
    bool custom_al = false;
    cudaStream_t stream = nullptr;
    lf_csr csr{};  // use_cell == 0: the caller's CSR (must outlive the handle)
    // lf_spmm on streams other than the build stream (lf_api.cu): each such
    // stream's last launch is recorded so lf_cell_destroy orders the free
    // after it, and counter slots reused across streams are fenced
    mutable std::mutex mu;
    mutable bool multi = false;
    mutable std::vector<std::pair<cudaStream_t, cudaEvent_t>> ext;
    mutable cudaEvent_t slot_ev[kCtrSlots] = {};
    float **dst_ring = nullptr;  // [kCtrSlots][lf::kMaxDst] destination bases of lf_spmm_ex, per counter slot
    mutable cudaStream_t slot_stream[kCtrSlots] = {};
    mutable bool slot_recorded[kCtrSlots] = {};
};
