// lf_api.cu -- the C ABI of liblf.so (include/liteform.h): argument checks,
// handle and memory management, the host side of configure (eq. 7 +
// Algorithm 3 over GPU statistics) and of the CSR -> CELL build.
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <string>
#include <mutex>
#include <vector>

#include "lf_internal.cuh"

namespace {

thread_local std::string g_detail;

lf_status fail(lf_status st, const std::string &why) {
    g_detail = why;
    return st;
}

#define LF_CUDA(expr)                                                                          \
    do {                                                                                       \
        cudaError_t e_ = (expr);                                                               \
        if (e_ != cudaSuccess) return fail(LF_ERR_CUDA, std::string(#expr) + ": " + cudaGetErrorString(e_)); \
    } while (0)

// ---- memory -------------------------------------------------------------
// Scratch (configure / build) and handles built without an lf_allocator come
// from a PRIVATE stream-ordered pool per device (cudaMemPoolCreate), not the
// device's default pool: its release threshold is raised so memory survives
// the synchronisations inside configure / build (a re-map costs
// milliseconds), but bounded, and no other cudaMallocAsync user of the
// process is affected.
constexpr uint64_t kPoolKeepBytes = uint64_t(512) << 20;
cudaMemPool_t scratch_pool() {
    static std::mutex mu;
    static cudaMemPool_t pools[64] = {};
    const int dev = lf::current_device();
    std::lock_guard<std::mutex> g(mu);
    if (!pools[dev]) {
        cudaMemPoolProps pr{};
        pr.allocType = cudaMemAllocationTypePinned;
        pr.handleTypes = cudaMemHandleTypeNone;
        pr.location.type = cudaMemLocationTypeDevice;
        pr.location.id = dev;
        cudaMemPool_t p = nullptr;
        if (cudaMemPoolCreate(&p, &pr) != cudaSuccess) return nullptr;
        uint64_t thr = kPoolKeepBytes;
        cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
        pools[dev] = p;
    }
    return pools[dev];
}
cudaError_t pool_alloc(void **p, size_t bytes, cudaStream_t s) {
    cudaMemPool_t pool = scratch_pool();
    if (!pool) return cudaErrorMemoryAllocation;
    return cudaMallocFromPoolAsync(p, bytes, pool, s);
}

struct Mem {
    const lf_allocator *al;
    cudaStream_t s;
    void *get(size_t bytes) {
        if (bytes == 0) return nullptr;
        bytes = (bytes + 255) & ~size_t(255);
        if (al && al->alloc) return al->alloc(al->ctx, bytes, s);
        void *p = nullptr;
        if (pool_alloc(&p, bytes, s) != cudaSuccess) return nullptr;
        return p;
    }
    void put(void *p, size_t bytes) {
        if (!p) return;
        bytes = (bytes + 255) & ~size_t(255);
        if (al && al->free) al->free(al->ctx, p, bytes, s);
        else cudaFreeAsync(p, s);
    }
};

// RAII list of allocations released at scope exit (scratch)
struct Scratch {
    Mem m;
    std::vector<std::pair<void *, size_t>> v;
    template <typename T>
    T *get(size_t n) {
        void *p = m.get(n * sizeof(T));
        if (n && p) v.push_back({p, n * sizeof(T)});
        return static_cast<T *>(p);
    }
    ~Scratch() {
        for (auto &x : v) m.put(x.first, x.second);
    }
};

lf_status check_csr(const lf_csr *A) {
    if (!A) return fail(LF_ERR_INVALID_ARG, "A is NULL");
    if (A->n_rows < 0 || A->n_cols < 0 || A->nnz < 0) return fail(LF_ERR_INVALID_ARG, "negative size");
    if (!A->row_ptr) return fail(LF_ERR_INVALID_ARG, "row_ptr is NULL");
    if (A->nnz > 0 && (!A->col_ind || !A->val)) return fail(LF_ERR_INVALID_ARG, "col_ind/val NULL with nnz > 0");
    if (A->n_cols > 2147483647LL) return fail(LF_ERR_INDEX_OVERFLOW, "n_cols exceeds int32");
    if (A->n_rows >= (int64_t(1) << 28)) return fail(LF_ERR_INDEX_OVERFLOW, "n_rows >= 2^28");
    return LF_OK;
}

lf_status maybe_validate(const lf_csr *A, cudaStream_t s) {
    const char *v = std::getenv("LF_VALIDATE");
    if (!v || v[0] != '1' || A->n_rows == 0) return LF_OK;
    int *d_flag = nullptr;
    LF_CUDA(pool_alloc(reinterpret_cast<void **>(&d_flag), sizeof(int), s));
    LF_CUDA(cudaMemsetAsync(d_flag, 0, sizeof(int), s));
    LF_CUDA(lf::launch_validate(*A, d_flag, s));
    int flag = 0;
    LF_CUDA(cudaMemcpyAsync(&flag, d_flag, sizeof(int), cudaMemcpyDeviceToHost, s));
    LF_CUDA(cudaFreeAsync(d_flag, s));
    LF_CUDA(cudaStreamSynchronize(s));
    if (flag & 2) return fail(LF_ERR_INVALID_ARG, "column index out of range or row_ptr decreasing");
    if (flag & 1) return fail(LF_ERR_UNSORTED_CSR, "columns not sorted within a row");
    return LF_OK;
}

// Table 2 + Table 3's J from the row-length sums
void table2_features(const lf_csr &A, int32_t J, const lf::StatsDev &st, double f[8]) {
    const double I = (double)A.n_rows;
    const double mean = A.n_rows ? (double)st.len_sum / I : 0.0;
    const double var = A.n_rows ? (double)st.len_sumsq / I - mean * mean : 0.0;
    f[0] = I;
    f[1] = (double)A.n_cols;
    f[2] = (double)st.len_sum;
    f[3] = mean;
    f[4] = A.n_rows ? (double)st.len_min : 0.0;
    f[5] = (double)st.len_max;
    f[6] = var > 0 ? std::sqrt(var) : 0.0;
    f[7] = (double)J;
}

// Grouped SpMM path (cell_spmm.cu): worth it when consecutive rows share
// many of their columns and the rows are long enough for a group to amortise
// the column merge.  Measured on B200 (per-slot -> grouped ms, J = 64 / 128):
// banded hw 4/8/12 (ratio 0.33-0.28) 1.06-1.8x faster, 32-wide dense blocks
// (0.25) 1.8-2.0x, 27-point stencil (0.50) 1.2x; slower on R-MAT (0.96),
// lognormal (~1), uniform (1.0, equal at J = 128) and rows of 8 (0.25, mean 8).
constexpr double kTcMaxSpan = 256.0;   // mean sampled window (B rows per 128-row group)
constexpr double kTcMaxOver = 0.02;    // sampled groups whose window exceeds the kernel's cap
constexpr double kGroupedMaxRatio = 0.6;    // distinct columns / nonzeros of 4-row groups
constexpr double kGroupedMinMeanLen = 8.5;  // mean row length
double group_ratio(const lf::StatsDev &st) {
    return st.grp_nnz ? (double)st.grp_union / (double)st.grp_nnz : 1.0;
}
bool grouped_candidate(const lf::StatsDev &st, const lf_csr &A, int32_t J) {
    const double mean = A.n_rows ? (double)st.len_sum / (double)A.n_rows : 0.0;
    return J <= 128 && st.grp_nnz > 0 && group_ratio(st) <= kGroupedMaxRatio && mean >= kGroupedMinMeanLen;
}

// Algorithm 3 in exponent space (reading R8) over eq. 7 costs.
int alg3(const int64_t *cost, int hi) {
    int lo = 0;
    while (lo < hi) {
        int mid = (lo + hi) / 2;
        if (cost[mid] > cost[mid + 1]) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

// SpMM kernel arguments of a handle (the counter slot is set per launch)
lf::SpmmArgs spmm_args(const lf_cell *h, const float *B, int64_t ldb, int32_t J, float *C, int64_t ldc) {
    const int nb = (int)h->buckets.size();
    lf::SpmmArgs a{h->d_buckets + nb, h->d_buckets + nb + h->nb_n, h->nb_n, h->nb_w, h->n_tasks_n, h->n_tasks_w,
                   h->slots_n, h->slots_w, 0, h->row_mode, h->n_rows, h->run_bound, nullptr, h->col_ind, h->val,
                   h->row_tag, B, ldb, C, ldc, J,
                   h->d_buckets + nb + h->nb_n + h->nb_w, h->nb_g, h->grouped, h->n_groups,
                   h->d_buckets + nb + h->nb_n + h->nb_w + h->nb_g, h->mma, h->n_groups_m,
                   h->d_buckets + nb + h->nb_n + h->nb_w + 2 * h->nb_g, h->nb_g, h->tc, h->n_groups_t, h->tc_win,
                   0, nullptr, 0, (uintptr_t)C};
    if (const char *g = std::getenv("LF_GROUPED")) a.grouped = g[0] == '1';
    if (const char *g = std::getenv("LF_TC")) a.tc = g[0] == '1';
    if (const char *g = std::getenv("LF_MMA")) a.mma = g[0] == '1';
    return a;
}

}  // namespace

// Entry of every call that launches work: a non-sticky CUDA error left
// pending by earlier, unrelated runtime calls of the process (cudaGetLastError
// reports the LAST error of the thread) is cleared here, so the status of
// this call reflects its own launches only.  A sticky error (a faulted
// context) is not cleared by this and fails the call's first launch.
static void clear_stale_error() { (void)cudaGetLastError(); }

extern "C" {

int32_t lf_abi_version(void) { return LF_ABI_VERSION; }

const char *lf_status_string(lf_status st) {
    switch (st) {
    case LF_OK: return "LF_OK";
    case LF_ERR_INVALID_ARG: return "LF_ERR_INVALID_ARG";
    case LF_ERR_UNSORTED_CSR: return "LF_ERR_UNSORTED_CSR";
    case LF_ERR_INDEX_OVERFLOW: return "LF_ERR_INDEX_OVERFLOW";
    case LF_ERR_NO_MEMORY: return "LF_ERR_NO_MEMORY";
    case LF_ERR_CUDA: return "LF_ERR_CUDA";
    case LF_ERR_UNSUPPORTED: return "LF_ERR_UNSUPPORTED";
    }
    return "LF_ERR_UNKNOWN";
}

const char *lf_last_error_detail(void) { return g_detail.c_str(); }

lf_status lf_cell_configure(const lf_csr *A, int32_t J, const lf_configure_opts *opts, lf_cell_params *out,
                            lf_configure_stats *stats, lf_stream_t stream) {
    g_detail.clear();
    clear_stale_error();
    if (lf_status st = check_csr(A)) return st;
    if (!out) return fail(LF_ERR_INVALID_ARG, "out is NULL");
    if (J < 1) return fail(LF_ERR_INVALID_ARG, "J < 1");
    lf_configure_opts o{};
    if (opts) o = *opts;
    if (o.max_parts < 0 || o.max_parts > LF_MAX_PARTS) return fail(LF_ERR_INVALID_ARG, "max_parts out of range");
    if (o.block_mult_log2 < 0 || o.block_mult_log2 > LF_MAX_LOG2) return fail(LF_ERR_INVALID_ARG, "block_mult_log2");
    if (o.force_parts < 0 || o.force_parts > LF_MAX_PARTS) return fail(LF_ERR_INVALID_ARG, "force_parts");
    if (o.force_width_log2 > LF_MAX_LOG2) return fail(LF_ERR_INVALID_ARG, "force_width_log2");
    if (o.force_format < 0 || o.force_format > 2) return fail(LF_ERR_INVALID_ARG, "force_format");
    const int max_parts = o.max_parts ? o.max_parts : LF_MAX_PARTS;
    cudaStream_t s = (cudaStream_t)stream;
    if (lf_status st = maybe_validate(A, s)) return st;

    // pinned staging buffer (one per thread) so the copies back are plain DMAs
    thread_local lf::StatsDev *h_st = nullptr;
    if (!h_st) LF_CUDA(cudaMallocHost(&h_st, sizeof(lf::StatsDev)));
    // GPU statistics for P partitions (one scratch allocation: stats, column
    // masks, per-segment t0 + mark tiles), copied back with one sync
    bool sampled = false;  // group / window samples already in h_st (they do not depend on P)
    auto run_stats = [&](int P) -> lf_status {
        const unsigned long long keep[5] = {h_st->grp_union, h_st->grp_nnz, h_st->win_span, h_st->win_cnt,
                                            h_st->win_over};
        const bool sample = !sampled;
        const size_t st_bytes = lf::stats_bytes(P);
        const size_t words = A->n_cols > 0 ? lf::mask_slots(A->n_cols) : 0;
        const size_t b_st = (st_bytes + 255) & ~size_t(255), b_mask = (words * 4 + 255) & ~size_t(255);
        const size_t b_t0 = A->n_rows > 0 ? lf::stats_scratch_bytes(A->n_rows, A->nnz, P) : 0;
        char *d = nullptr;
        LF_CUDA(pool_alloc(reinterpret_cast<void **>(&d), b_st + b_mask + b_t0 + 256, s));
        lf::StatsDev *d_st = reinterpret_cast<lf::StatsDev *>(d);
        uint32_t *d_mask = words ? reinterpret_cast<uint32_t *>(d + b_st) : nullptr;
        uint8_t *d_t0 = b_t0 ? reinterpret_cast<uint8_t *>(d + b_st + b_mask) : nullptr;
        // stats and masks are adjacent: one memset zeroes both
        LF_CUDA(cudaMemsetAsync(d, 0, b_st + b_mask, s));
        LF_CUDA(cudaMemsetAsync(&d_st->len_min, 0xFF, sizeof(unsigned long long), s));
        LF_CUDA(lf::launch_stats(*A, P, d_st, d_mask, d_t0, s, sample));
        LF_CUDA(cudaMemcpyAsync(h_st, d_st, st_bytes, cudaMemcpyDeviceToHost, s));
        LF_CUDA(cudaFreeAsync(d, s));
        LF_CUDA(cudaStreamSynchronize(s));
        if (!sample) {
            h_st->grp_union = keep[0];
            h_st->grp_nnz = keep[1];
            h_st->win_span = keep[2];
            h_st->win_cnt = keep[3];
            h_st->win_over = keep[4];
        }
        sampled = true;
        return LF_OK;
    };
    // predictor (sections 5.1-5.2): it needs the Table 2 row-length features
    // before P is known.  The statistics pass computes them too, so for
    // matrices up to kSpeculateNnz nonzeros it runs once speculatively for
    // P = 1 (the forced P if given) and again only if the predictor picks
    // another P: one pass and one sync in the common case.  Larger matrices
    // (where a wasted pass costs more than a sync) read the features from
    // row_ptr alone first.
    constexpr int64_t kSpeculateNnz = int64_t(1) << 25;
    int P = o.force_parts ? o.force_parts : 1;
    int use_cell = o.force_format == 2 ? 0 : 1;
    const bool predict = o.force_parts == 0 || o.force_format == 0;
    bool have = false;
    if (predict) {
        if (o.force_parts != 0 || A->nnz <= kSpeculateNnz) {
            if (lf_status st = run_stats(P)) return st;
            have = true;
        } else {
            lf::StatsDev *d_f = nullptr;
            const size_t fb = lf::stats_bytes(0);
            LF_CUDA(pool_alloc(reinterpret_cast<void **>(&d_f), fb, s));
            LF_CUDA(cudaMemsetAsync(d_f, 0, fb, s));
            LF_CUDA(cudaMemsetAsync(&d_f->len_min, 0xFF, sizeof(unsigned long long), s));
            LF_CUDA(lf::launch_features(*A, d_f, s));
            LF_CUDA(cudaMemcpyAsync(h_st, d_f, fb, cudaMemcpyDeviceToHost, s));
            LF_CUDA(cudaFreeAsync(d_f, s));
            LF_CUDA(cudaStreamSynchronize(s));
            sampled = A->n_rows >= lf::kGroupRows && A->nnz > 0;
        }
        double f[8];
        table2_features(*A, J, *h_st, f);
        int32_t pu = 1, pp = 1;
        if (lf_status st = lf_predict(f, max_parts, &pu, &pp)) return fail(st, "lf_predict");
        if (o.force_format == 0) use_cell = pu;
        // the grouped CELL path (not in the paper's label space, trained on
        // the per-slot kernel) beats the CSR kernel where it applies: keep
        // CELL then (measured: 27-point stencil 0.82 vs 0.98 ms at J = 64)
        if (o.force_format == 0 && !pu && grouped_candidate(*h_st, *A, J)) use_cell = 1;
        if (o.force_parts == 0 && pp != P) {
            P = pp;
            have = false;
        }
    }
    // the fixed CSR format needs no CELL composition (section 5: the
    // predictor picks the format first): no statistics pass then
    const bool need_stats = use_cell != 0;
    if (!have && need_stats)
        if (lf_status st = run_stats(P)) return st;
    if (!have && !need_stats && !predict) {  // forced CSR: the features alone
        lf::StatsDev *d_f = nullptr;
        const size_t fb = lf::stats_bytes(0);
        LF_CUDA(pool_alloc(reinterpret_cast<void **>(&d_f), fb, s));
        LF_CUDA(cudaMemsetAsync(d_f, 0, fb, s));
        LF_CUDA(cudaMemsetAsync(&d_f->len_min, 0xFF, sizeof(unsigned long long), s));
        LF_CUDA(lf::launch_features(*A, d_f, s));
        LF_CUDA(cudaMemcpyAsync(h_st, d_f, fb, cudaMemcpyDeviceToHost, s));
        LF_CUDA(cudaFreeAsync(d_f, s));
        LF_CUDA(cudaStreamSynchronize(s));
    }
    if (!have && !need_stats) std::memset(h_st->part, 0, sizeof(h_st->part[0]) * (size_t)P);
    const lf::StatsDev &st = *h_st;

    lf_configure_stats local;
    lf_configure_stats &cs = stats ? *stats : local;
    std::memset(&cs, 0, sizeof(cs));
    table2_features(*A, J, st, cs.features);
    cs.n_parts = P;

    lf_cell_params prm{};
    prm.use_cell = use_cell;
    prm.n_parts = P;
    for (int p = 0; p < P; p++) {
        int top = -1;
        for (int t = 0; t < lf::kMaxT; t++) {
            cs.H[p][t] = (int64_t)st.part[p].H[t];
            cs.F[p][t] = (int64_t)st.part[p].F[t];
            cs.Unat[p][t] = (int64_t)st.part[p].Unat[t];
            cs.Utop[p][t] = (int64_t)st.part[p].Utop[t];
            cs.cost[p][t] = -1;
            if (st.part[p].H[t]) top = t;
        }
        cs.max_log2[p] = top;
        // eq. 7 (reading R10): buckets b < e keep their natural rows,
        // the max bucket e holds every row with ceil_log2 l >= e, folded.
        for (int e = 0; e <= top; e++) {
            int64_t c = 0;
            for (int b = 0; b < e; b++)
                if (cs.H[p][b]) c += 2 * cs.H[p][b] * (int64_t(1) << b) + cs.Unat[p][b] * J + cs.H[p][b] * J;
            if (cs.F[p][e]) c += 2 * cs.F[p][e] * (int64_t(1) << e) + cs.Utop[p][e] * J + cs.F[p][e] * J;
            cs.cost[p][e] = c;
        }
        int e;
        if (top < 0) e = 0;
        else if (o.force_width_log2 >= 0) e = std::min(o.force_width_log2, top);
        else e = alg3(cs.cost[p], top);
        cs.chosen_log2[p] = top < 0 ? -1 : e;
        prm.max_width_log2[p] = (int8_t)e;
        prm.block_nnz_log2[p] = (int8_t)std::min(e + o.block_mult_log2, LF_MAX_LOG2);
    }
    // grouped SpMM path (cell_spmm.cu): worth it when consecutive rows share
    // most of their columns and the rows are long enough for a group to
    // amortise the column merge (measured on B200: banded / dense-block rows
    // of 25-32 nonzeros at ratio <= 0.28 gain 1.3-1.45x, the 27-point stencil
    // at 0.50 and rows of 8 lose); needs every W_p <= 32 and J <= 128
    cs.group_union_ratio = group_ratio(st);
    bool narrow = true;
    for (int p = 0; p < P; p++) narrow = narrow && prm.max_width_log2[p] <= 5;
    cs.spmm_grouped = (use_cell && narrow && grouped_candidate(st, *A, J)) ? 1 : 0;
    // tcgen05 windowed path (cell_spmm_tc.cu): groups of 128 rows whose
    // columns fit a window of <= 256 B rows, the window short enough that
    // the dense contraction (3 MMAs per 8 window rows) stays under the group's
    // memory time; decided from the sampled windows
    cs.window_span_mean = st.win_cnt ? (double)st.win_span / (double)st.win_cnt : 0.0;
    cs.window_over_frac = st.win_cnt ? (double)st.win_over / (double)st.win_cnt : 1.0;
    cs.spmm_tc = (use_cell && narrow && J >= 32 && J <= 128 && st.win_cnt > 0 && cs.window_over_frac <= kTcMaxOver &&
                  cs.window_span_mean <= kTcMaxSpan)
                     ? 1
                     : 0;
    *out = prm;
    return LF_OK;
}

lf_status lf_cell_build(const lf_csr *A, const lf_cell_params *params, const lf_configure_stats *stats,
                        const lf_allocator *al, lf_stream_t stream, lf_cell **out) {
    g_detail.clear();
    clear_stale_error();
    if (lf_status st = check_csr(A)) return st;
    if (!params || !out) return fail(LF_ERR_INVALID_ARG, "params/out is NULL");
    *out = nullptr;
    const int P = params->n_parts;
    if (P < 1 || P > LF_MAX_PARTS) return fail(LF_ERR_INVALID_ARG, "n_parts out of range");
    if (params->use_cell != 0 && params->use_cell != 1) return fail(LF_ERR_INVALID_ARG, "use_cell");
    for (int p = 0; p < P; p++) {
        const int e = params->max_width_log2[p], k = params->block_nnz_log2[p];
        if (e < 0 || e > LF_MAX_LOG2 || k < e || k > LF_MAX_LOG2)
            return fail(LF_ERR_INVALID_ARG, "need 0 <= e_p <= k_p <= 30");
    }
    if (al && (!al->alloc || !al->free)) return fail(LF_ERR_INVALID_ARG, "allocator without alloc/free");
    if (stats) {  // the bucket sizes come from the stats: they must describe THIS A at this P
        if (stats->n_parts != P) return fail(LF_ERR_INVALID_ARG, "stats were computed for another n_parts");
        if (stats->features[0] != (double)A->n_rows || stats->features[1] != (double)A->n_cols ||
            stats->features[2] != (double)A->nnz)
            return fail(LF_ERR_INVALID_ARG, "stats were computed for another matrix (n_rows / n_cols / nnz differ)");
        // F[p][0] = sum of the segment lengths of partition p, so the F[.][0]
        // column sums to nnz exactly; tables zeroed by a CSR-format configure
        // (or a stale / foreign struct) fail this
        int64_t f0 = 0;
        for (int p = 0; p < P; p++) {
            f0 += stats->F[p][0];
            for (int t = 0; t < lf::kMaxT; t++)
                if (stats->H[p][t] < 0 || stats->F[p][t] < 0) return fail(LF_ERR_INVALID_ARG, "negative stats table entry");
        }
        if (f0 != A->nnz)
            return fail(LF_ERR_INVALID_ARG, "stats tables do not cover A (sum of F[p][0] != nnz): configure chose "
                                            "the CSR format or the stats belong to another matrix");
    }
    cudaStream_t s = (cudaStream_t)stream;
    if (lf_status st = maybe_validate(A, s)) return st;

    lf_cell *h = new lf_cell();
    h->params = *params;
    h->grouped = stats ? stats->spmm_grouped : 0;
    h->tc = stats ? stats->spmm_tc : 0;
    h->n_rows = A->n_rows;
    h->n_cols = A->n_cols;
    h->nnz = A->nnz;
    h->stream = s;
    if (al) {
        h->al = *al;
        h->custom_al = true;
    }
    auto bail = [&](lf_status st) {
        lf_cell_destroy(h);
        return st;
    };
    if (params->use_cell == 0) {  // fixed format: keep the caller's CSR
        h->csr = *A;
        *out = h;
        return LF_OK;
    }
    Mem mem{al, s};
    const int64_t I = A->n_rows;
    const int n_tiles = (int)((I + lf::kBuildTile - 1) / lf::kBuildTile);
    auto cu = [&](cudaError_t e, const char *what) -> lf_status {
        if (e != cudaSuccess) return fail(LF_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
        return LF_OK;
    };
    lf_status st;
    lf::BuildScratch bs{};
    bs.n_tiles = n_tiles;
    lf::WidthArg e_arg{};
    for (int p = 0; p < P; p++) e_arg.e[p] = params->max_width_log2[p];

    // host: bucket table (R2, R7) and warp-task decomposition from the bucket
    // sizes (CELL rows per (p, t))
    int64_t R_tot = 0, S_tot = 0;
    std::vector<long long> row_off((size_t)P * lf::kMaxT, -1);
    auto make_table = [&](const std::vector<long long> &tot) -> lf_status {
        std::vector<lf::BucketDev> bn, bw;
        for (int p = 0; p < P; p++) {
            const int k = params->block_nnz_log2[p];
            for (int t = 0; t <= params->max_width_log2[p]; t++) {
                const long long n = tot[(size_t)p * lf::kMaxT + t];
                if (n == 0) continue;
                const int64_t R = int64_t(1) << (k - t), W = int64_t(1) << t;
                const int64_t pad = (n + R - 1) / R * R;
                lf_bucket b{};
                b.part = p;
                b.width_log2 = t;
                b.rows_per_block = (int32_t)std::min<int64_t>(R, INT32_MAX);
                b.n_rows = n;
                b.n_rows_pad = pad;
                b.row_off = R_tot;
                b.slot_off = S_tot;
                h->buckets.push_back(b);
                lf::BucketDev d{};
                d.slot_off = S_tot;
                d.row_off = R_tot;
                d.n_slots = pad * W;
                d.n_real_rows = n;
                d.n_rows_pad = pad;
                d.t = t;
                d.piece_log2 = std::max(0, t - lf::kPieceLog2);
                d.task_slots = (int32_t)std::max<int64_t>(32, W >> d.piece_log2);
                if (W < 32) {
                    d.task_off = h->n_tasks_n;
                    h->n_tasks_n += (pad * W + 31) / 32;
                    h->slots_n += pad * W;
                    bn.push_back(d);
                } else {
                    d.task_off = h->n_tasks_w;
                    h->n_tasks_w += pad << d.piece_log2;
                    h->slots_w += pad * W;
                    bw.push_back(d);
                }
                d.task_off = 0;
                h->h_buckets.push_back(d);
                row_off[(size_t)p * lf::kMaxT + t] = R_tot;
                R_tot += pad;
                S_tot += pad * W;
            }
        }
        h->n_cell_rows = R_tot;
        h->n_slots = S_tot;
        h->nb_n = (int)bn.size();
        h->nb_w = (int)bw.size();
        const int nb_all = (int)h->h_buckets.size();
        h->h_buckets.insert(h->h_buckets.end(), bn.begin(), bn.end());
        h->h_buckets.insert(h->h_buckets.end(), bw.begin(), bw.end());
        // grouped SpMM path (every W <= 32): the buckets again, task_off
        // counting groups of kGroupRows CELL rows
        bool narrow = nb_all > 0;
        for (int q = 0; q < nb_all; q++) narrow = narrow && h->h_buckets[q].t <= 5;
        if (narrow) {
            for (int q = 0; q < nb_all; q++) {
                lf::BucketDev d = h->h_buckets[q];
                d.task_off = h->n_groups;
                h->n_groups += (d.n_rows_pad + lf::kGroupRows - 1) / lf::kGroupRows;
                h->h_buckets.push_back(d);
            }
            for (int q = 0; q < nb_all; q++) {  // and again for 16-row groups (tensor-core path)
                lf::BucketDev d = h->h_buckets[q];
                d.task_off = h->n_groups_m;
                h->n_groups_m += (d.n_rows_pad + 15) / 16;
                h->h_buckets.push_back(d);
            }
            for (int q = 0; q < nb_all; q++) {  // and for 128-row groups (tcgen05 windowed path)
                lf::BucketDev d = h->h_buckets[q];
                d.task_off = h->n_groups_t;
                h->n_groups_t += (d.n_rows_pad + lf::kTcGroupRows - 1) / lf::kTcGroupRows;
                h->h_buckets.push_back(d);
            }
            h->nb_g = nb_all;
        }
        if (h->buckets.size() > 2048) return fail(LF_ERR_UNSUPPORTED, "more than 2048 buckets");
        return LF_OK;
    };

    // scratch, ONE allocation: [seg_rel | tile_cnt | key_total | row_cnt | src_pos | src_cnt]
    // (src_* sized by R_tot: known up front when the configure stats are passed)
    const size_t a256 = 256;
    auto up = [&](size_t b) { return (b + a256 - 1) / a256 * a256; };
    const size_t s_seg = P > 1 ? up((size_t)I * (P - 1) * 4) : 0,
                 s_tc = up((size_t)P * lf::kMaxT * std::max(n_tiles, 1) * 8), s_kt = up((size_t)P * lf::kMaxT * 8),
                 s_rc = up((size_t)std::max<int64_t>(I, 1) * 4);
    const size_t s_head = s_seg + s_tc + s_kt + s_rc;
    // build-time scratch comes from the device's stream-ordered pool (as the
    // configure scratch): no allocator callback into the caller's runtime for
    // memory that lives only until the end of this call
    Scratch sc{Mem{nullptr, s}, {}};
    std::vector<long long> tot((size_t)P * lf::kMaxT, 0);
    if (stats) {  // bucket sizes from the configure statistics: no synchronisation
        for (int p = 0; p < P; p++) {
            const int e = params->max_width_log2[p];
            for (int t = 0; t < e && t < lf::kMaxT; t++) tot[(size_t)p * lf::kMaxT + t] = stats->H[p][t];
            if (e < lf::kMaxT) tot[(size_t)p * lf::kMaxT + e] = stats->F[p][e];
        }
        if ((st = make_table(tot))) return bail(st);
    }
    const size_t s_src = stats ? up((size_t)R_tot * 8) + up((size_t)R_tot * 4) : 0;
    char *scr = sc.get<char>(s_head + s_src);
    if (!scr) return bail(fail(LF_ERR_NO_MEMORY, "scratch allocation failed"));
    bs.seg_rel = P > 1 ? reinterpret_cast<int32_t *>(scr) : nullptr;
    bs.tile_cnt = reinterpret_cast<long long *>(scr + s_seg);
    bs.key_total = reinterpret_cast<long long *>(scr + s_seg + s_tc);
    int32_t *row_cnt = reinterpret_cast<int32_t *>(scr + s_seg + s_tc + s_kt);

    // a1 + a4 (count): segments, bucket keys, per-tile totals, tile scan
    // (P = 1: bucket_kernel<0> writes every row_cnt entry itself)
    if (P > 1 && I > 0 &&
        (st = cu(cudaMemsetAsync(row_cnt, 0, (size_t)I * sizeof(int32_t), s), "memset")))
        return bail(st);
    if ((st = cu(lf::launch_seg(*A, P, bs.seg_rel, s), "seg"))) return bail(st);
    if ((st = cu(lf::launch_bucket_count(*A, P, e_arg, bs, row_cnt, s), "bucket_count"))) return bail(st);
    if (n_tiles > 0 && (st = cu(lf::launch_tile_scan(P, bs, s), "tile_scan"))) return bail(st);
    if (!stats) {
        if (n_tiles > 0 &&
            (st = cu(cudaMemcpyAsync(tot.data(), bs.key_total, tot.size() * 8, cudaMemcpyDeviceToHost, s), "D2H")))
            return bail(st);
        if ((st = cu(cudaStreamSynchronize(s), "sync"))) return bail(st);
        if ((st = make_table(tot))) return bail(st);
        char *src = sc.get<char>(up((size_t)R_tot * 8) + up((size_t)R_tot * 4));
        if (R_tot && !src) return bail(fail(LF_ERR_NO_MEMORY, "scratch allocation failed"));
        bs.src_pos = reinterpret_cast<int64_t *>(src);
        bs.src_cnt = R_tot ? reinterpret_cast<int32_t *>(src + up((size_t)R_tot * 8)) : nullptr;
    } else {
        bs.src_pos = reinterpret_cast<int64_t *>(scr + s_head);
        bs.src_cnt = reinterpret_cast<int32_t *>(scr + s_head + up((size_t)R_tot * 8));
        const char *v = std::getenv("LF_VALIDATE");
        if (v && v[0] == '1' && n_tiles > 0) {  // the GPU-counted bucket sizes must equal the stats' ones
            std::vector<long long> cnt(tot.size(), 0);
            if ((st = cu(cudaMemcpyAsync(cnt.data(), bs.key_total, cnt.size() * 8, cudaMemcpyDeviceToHost, s), "D2H")))
                return bail(st);
            if ((st = cu(cudaStreamSynchronize(s), "sync"))) return bail(st);
            if (cnt != tot) return bail(fail(LF_ERR_INVALID_ARG, "bucket sizes counted on the GPU differ from the stats"));
        }
    }
    const int nb = (int)h->buckets.size();

    // persistent arrays, ONE allocation (the pool): a header copied with one
    // H2D [bucket table | key_row_off], then rowInd, row tags, colInd, val,
    // run bounds, queue counters, row modes
    const size_t b_bk = up(h->h_buckets.size() * sizeof(lf::BucketDev)), b_ko = up(row_off.size() * 8),
                 b_ri = up(R_tot * 4), b_rt = up(R_tot * 4), b_ci = up(S_tot * 4), b_va = up(S_tot * 4),
                 b_rb = up((size_t)(h->n_tasks_w + 1)), b_ct = up(kCtrSlots * 4 * sizeof(unsigned long long)),
                 b_rm = up((size_t)std::max<int64_t>(I, 1));
    // tcgen05 windowed path: a window per 128-row group, built when configure
    // chose the path (or LF_TC=1 asks for it, or the sizes are GPU-counted)
    const char *tc_env = std::getenv("LF_TC");
    const bool want_tc = h->nb_g > 0 && h->n_groups_t > 0 &&
                         (tc_env ? tc_env[0] == '1' : (stats ? stats->spmm_tc != 0 : true));
    const size_t b_tw = want_tc ? up((size_t)h->n_groups_t * sizeof(int2)) : 0;
    const size_t b_dr = up((size_t)kCtrSlots * lf::kMaxDst * sizeof(float *));
    h->pool_bytes = b_bk + b_ko + b_ri + b_rt + b_ci + b_va + b_rb + b_ct + b_rm + b_tw + b_dr;
    h->pool = mem.get(h->pool_bytes);
    if (!h->pool) return bail(fail(LF_ERR_NO_MEMORY, "CELL arrays allocation failed"));
    char *q = static_cast<char *>(h->pool);
    h->d_buckets = reinterpret_cast<lf::BucketDev *>(q);
    bs.key_row_off = reinterpret_cast<long long *>(q + b_bk);
    q += b_bk + b_ko;
    h->row_ind = reinterpret_cast<int32_t *>(q);
    h->row_tag = reinterpret_cast<int32_t *>(q + b_ri);
    h->col_ind = reinterpret_cast<int32_t *>(q + b_ri + b_rt);
    h->val = reinterpret_cast<float *>(q + b_ri + b_rt + b_ci);
    h->run_bound = reinterpret_cast<uint8_t *>(q + b_ri + b_rt + b_ci + b_va);
    h->ctr_ring = reinterpret_cast<unsigned long long *>(q + b_ri + b_rt + b_ci + b_va + b_rb);
    h->row_mode = reinterpret_cast<uint8_t *>(q + b_ri + b_rt + b_ci + b_va + b_rb + b_ct);
    h->tc_win = b_tw ? reinterpret_cast<int2 *>(q + b_ri + b_rt + b_ci + b_va + b_rb + b_ct + b_rm) : nullptr;
    h->dst_ring = reinterpret_cast<float **>(q + b_ri + b_rt + b_ci + b_va + b_rb + b_ct + b_rm + b_tw);
    {
        std::vector<char> head(b_bk + b_ko, 0);
        if (!h->h_buckets.empty())
            std::memcpy(head.data(), h->h_buckets.data(), h->h_buckets.size() * sizeof(lf::BucketDev));
        std::memcpy(head.data() + b_bk, row_off.data(), row_off.size() * 8);
        if ((st = cu(cudaMemcpyAsync(h->pool, head.data(), head.size(), cudaMemcpyHostToDevice, s), "H2D table")))
            return bail(st);
    }
    // P > 1: several blocks update one row's mode, so it starts at kRowEmpty
    if (P > 1 && I > 0 && (st = cu(cudaMemsetAsync(h->row_mode, lf::kRowEmpty, (size_t)I, s), "memset")))
        return bail(st);
    // queue counters zero; padding rows' rowInd / tags -1 and src_cnt 0
    if ((st = cu(lf::launch_pad_init(h->d_buckets, nb, h->row_ind, h->row_tag, bs.src_cnt, bs.src_pos, h->ctr_ring,
                                     kCtrSlots * 4, s),
                 "pad_init")))
        return bail(st);
    // a4 (place) + a5 (scatter)
    if ((st = cu(lf::launch_bucket_place(*A, P, e_arg, bs, row_cnt, h->row_ind, h->row_tag, h->row_mode, s),
                 "bucket_place")))
        return bail(st);
    if ((st = cu(lf::launch_slot_fill(*A, h->d_buckets, nb, S_tot, bs, h->col_ind, h->val, s), "slot_fill")))
        return bail(st);
    if ((st = cu(lf::launch_run_bounds(h->d_buckets + nb + h->nb_n, h->nb_w, h->n_tasks_w, h->row_tag, h->run_bound,
                                       s),
                 "run_bounds")))
        return bail(st);
    if (h->tc_win &&
        (st = cu(lf::launch_tc_windows(h->d_buckets + nb + h->nb_n + h->nb_w + 2 * h->nb_g, h->nb_g, h->n_groups_t,
                                       h->col_ind, bs.src_cnt, h->tc_win, s),
                 "tc_windows")))
        return bail(st);

    *out = h;
    return LF_OK;
}

lf_status lf_spmm(const lf_cell *h, const float *B, int64_t ldb, int32_t J, float *C, int64_t ldc,
                  lf_stream_t stream) {
    return lf_spmm_ex(h, B, ldb, J, C, ldc, nullptr, stream);
}

lf_status lf_spmm_ex(const lf_cell *h, const float *B, int64_t ldb, int32_t J, float *C, int64_t ldc,
                     const lf_spmm_opts *opts, lf_stream_t stream) {
    g_detail.clear();
    clear_stale_error();
    if (!h) return fail(LF_ERR_INVALID_ARG, "handle is NULL");
    if (J < 0 || ldb < J || ldc < J || ldb < 0 || ldc < 0) return fail(LF_ERR_INVALID_ARG, "need 0 <= J <= ldb, ldc");
    const int n_dst = opts ? opts->n_dst : 0;
    if (n_dst < 0 || n_dst > LF_MAX_DST) return fail(LF_ERR_INVALID_ARG, "n_dst outside [0, LF_MAX_DST]");
    if (n_dst > 0) {
        if (!opts->dst) return fail(LF_ERR_INVALID_ARG, "dst is NULL");
        if (opts->row_base < 0) return fail(LF_ERR_INVALID_ARG, "row_base < 0");
        for (int d = 0; d < n_dst; d++)
            if (!opts->dst[d]) return fail(LF_ERR_INVALID_ARG, "a destination pointer is NULL");
    }
    if (J == 0 || h->n_rows == 0) return LF_OK;
    if (!C && n_dst == 0) return fail(LF_ERR_INVALID_ARG, "C is NULL");
    if (!B && h->n_cols > 0) return fail(LF_ERR_INVALID_ARG, "B is NULL");
    cudaStream_t s = (cudaStream_t)stream;
    if (h->params.use_cell == 0) {
        if (n_dst > 0) return fail(LF_ERR_UNSUPPORTED, "fused row exchange needs a CELL handle (use_cell = 1)");
        LF_CUDA(lf::launch_csr_spmm(h->csr, B, ldb, J, C, ldc, s));
        return LF_OK;
    }
    lf::SpmmArgs a = spmm_args(h, B, ldb, J, C, ldc);
    const uint32_t k = h->launch_seq.fetch_add(1, std::memory_order_relaxed) % kCtrSlots;
    a.ctr = h->ctr_ring + 4 * k;
    if (n_dst > 0) {  // the destinations travel in the launch's own slot of the handle's ring
        a.n_dst = n_dst;
        a.dst = h->dst_ring + (size_t)k * lf::kMaxDst;
        a.row_base = opts->row_base;
        a.c_bits = 0;
        for (int d = 0; d < n_dst; d++) a.c_bits |= (uintptr_t)opts->dst[d];
        LF_CUDA(cudaMemcpyAsync(h->dst_ring + (size_t)k * lf::kMaxDst, opts->dst, (size_t)n_dst * sizeof(float *),
                                cudaMemcpyHostToDevice, s));
    }
    std::lock_guard<std::mutex> g(h->mu);
    if (s == h->stream && !h->multi) {  // the common case: one stream, launches ordered by it
        LF_CUDA(lf::launch_cell_spmm(a, s));
        return LF_OK;
    }
    // several streams: a counter slot whose previous launch ran on another
    // stream is fenced behind it, and every stream's last launch is recorded
    // for lf_cell_destroy
    if (!h->multi) {  // every earlier launch ran on the build stream
        h->multi = true;
        for (int q = 0; q < kCtrSlots; q++) h->slot_stream[q] = h->stream;
    }
    if (h->slot_stream[k] != s) {
        if (!h->slot_ev[k]) LF_CUDA(cudaEventCreateWithFlags(&h->slot_ev[k], cudaEventDisableTiming));
        if (!h->slot_recorded[k])  // earlier launches of the build stream were not recorded
            LF_CUDA(cudaEventRecord(h->slot_ev[k], h->stream));
        LF_CUDA(cudaStreamWaitEvent(s, h->slot_ev[k], 0));
    }
    LF_CUDA(lf::launch_cell_spmm(a, s));
    if (!h->slot_ev[k]) LF_CUDA(cudaEventCreateWithFlags(&h->slot_ev[k], cudaEventDisableTiming));
    LF_CUDA(cudaEventRecord(h->slot_ev[k], s));
    h->slot_recorded[k] = true;
    h->slot_stream[k] = s;
    if (s != h->stream) {
        cudaEvent_t *e = nullptr;
        for (auto &x : h->ext)
            if (x.first == s) e = &x.second;
        if (!e) {
            h->ext.push_back({s, nullptr});
            e = &h->ext.back().second;
            LF_CUDA(cudaEventCreateWithFlags(e, cudaEventDisableTiming));
        }
        LF_CUDA(cudaEventRecord(*e, s));
    }
    return LF_OK;
}

const char *lf_spmm_kernel_name(const lf_cell *h, int32_t J) {
    if (!h || J <= 0) return "";
    if (h->params.use_cell == 0) return "csr_spmm_kernel";
    static const float *kAligned = reinterpret_cast<const float *>(uintptr_t(256));
    lf::SpmmArgs a = spmm_args(h, kAligned, J, J, const_cast<float *>(kAligned), J);
    return lf::cell_spmm_path(a);
}

lf_status lf_csr_spmm(const lf_csr *A, const float *B, int64_t ldb, int32_t J, float *C, int64_t ldc,
                      lf_stream_t stream) {
    g_detail.clear();
    clear_stale_error();
    if (lf_status st = check_csr(A)) return st;
    if (J < 0 || ldb < J || ldc < J) return fail(LF_ERR_INVALID_ARG, "need 0 <= J <= ldb, ldc");
    if (J == 0 || A->n_rows == 0) return LF_OK;
    if (!C || (!B && A->n_cols > 0)) return fail(LF_ERR_INVALID_ARG, "B/C is NULL");
    LF_CUDA(lf::launch_csr_spmm(*A, B, ldb, J, C, ldc, (cudaStream_t)stream));
    return LF_OK;
}

lf_status lf_cell_view(const lf_cell *h, lf_cell_arrays *out) {
    if (!h || !out) return fail(LF_ERR_INVALID_ARG, "NULL argument");
    std::memset(out, 0, sizeof(*out));
    out->n_rows = h->n_rows;
    out->n_cols = h->n_cols;
    out->nnz = h->nnz;
    out->n_cell_rows = h->n_cell_rows;
    out->n_slots = h->n_slots;
    out->n_buckets = (int32_t)h->buckets.size();
    out->row_ind = h->row_ind;
    out->col_ind = h->col_ind;
    out->val = h->val;
    out->buckets = h->buckets.empty() ? nullptr : h->buckets.data();
    out->params = h->params;
    return LF_OK;
}

lf_status lf_cell_destroy(lf_cell *h) {
    if (!h) return LF_OK;
    // the free is ordered on the build stream: after every lf_spmm launched on
    // another stream too (their last launches were recorded)
    for (auto &x : h->ext) {
        cudaStreamWaitEvent(h->stream, x.second, 0);
        cudaEventDestroy(x.second);
    }
    for (int q = 0; q < kCtrSlots; q++)
        if (h->slot_ev[q]) cudaEventDestroy(h->slot_ev[q]);
    Mem mem{h->custom_al ? &h->al : nullptr, h->stream};
    mem.put(h->pool, h->pool_bytes);
    delete h;
    return LF_OK;
}

}  // extern "C"
