// cell_stats.cu -- configure statistics on the GPU.
//
// One pass over the CSR produces, per partition p and natural bucket
// t = ceil_log2(l) of every non-empty row segment (reading R1):
//   H[p][t]  segment count,  F[p][t] = sum_{t0 >= t} ceil(l / 2^t)  (fold rows),
// the Table 2 row-length statistics, and a per-column bitmask
// M[c] |= 1 << t0 (the partition of column c is c / S).  A second pass over
// the K columns turns M into Unat[p][t] = #{c : bit t} and
// Utop[p][t] = #{c : highest bit >= t}: the |set(Ind)| terms of eq. 7
// for every candidate max width at once.
#include "../lf_internal.cuh"

namespace lf {

namespace {

constexpr int kThreads = 256;
constexpr int kLongSeg = 32;  // segments longer than this are marked warp-cooperatively

__device__ __forceinline__ int64_t lower_bound_col(const int32_t *__restrict__ col, int64_t b, int64_t e,
                                                   int64_t v) {
    while (b < e) {
        int64_t m = (b + e) >> 1;
        if (col[m] < v) b = m + 1;
        else e = m;
    }
    return b;
}

__device__ __forceinline__ void mark(uint32_t *mask, int32_t c, uint32_t bit) {
    // bits are only ever set, so a stale read just costs one extra atomic
    if (!(mask[c] & bit)) atomicOr(mask + c, bit);
}

__global__ void __launch_bounds__(kThreads) stats_rows_kernel(const int64_t *__restrict__ row_ptr,
                                                              const int32_t *__restrict__ col, int64_t n_rows,
                                                              int64_t S, int P, StatsDev *st, uint32_t *mask) {
    extern __shared__ unsigned long long sh[];  // H_s[P][32], F_s[P][32]
    unsigned long long *H_s = sh, *F_s = sh + P * kMaxT;
    for (int q = threadIdx.x; q < 2 * P * kMaxT; q += blockDim.x) sh[q] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    unsigned long long mn = ~0ull, mx = 0, sum = 0, sq = 0;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n_rows; base += stride) {
        const int64_t i = base + threadIdx.x;
        const bool active = i < n_rows;
        int64_t rb = 0, re = 0;
        if (active) {
            rb = row_ptr[i];
            re = row_ptr[i + 1];
            unsigned long long len = (unsigned long long)(re - rb);
            mn = min(mn, len);
            mx = max(mx, len);
            sum += len;
            sq += len * len;
        }
        int64_t b = rb;
        for (int p = 0; p < P; p++) {
            int64_t e = (p == P - 1) ? re : lower_bound_col(col, b, re, (int64_t)(p + 1) * S);
            int64_t l = e - b;
            int t0 = 0;
            if (l > 0) {
                t0 = ceil_log2_i64(l);
                atomicAdd(&H_s[p * kMaxT + t0], 1ull);
                for (int t = 0; t <= t0; t++)
                    atomicAdd(&F_s[p * kMaxT + t], (unsigned long long)((l + (int64_t(1) << t) - 1) >> t));
                if (l <= kLongSeg)
                    for (int64_t q = b; q < e; q++) mark(mask, col[q], 1u << t0);
            }
            // long segments: the whole warp marks them together
            unsigned long_lanes = __ballot_sync(0xffffffffu, l > kLongSeg);
            while (long_lanes) {
                int src = __ffs(long_lanes) - 1;
                long_lanes &= long_lanes - 1;
                int64_t sb = __shfl_sync(0xffffffffu, b, src);
                int64_t se = __shfl_sync(0xffffffffu, e, src);
                int st0 = __shfl_sync(0xffffffffu, t0, src);
                for (int64_t q = sb + lane; q < se; q += 32) mark(mask, col[q], 1u << st0);
            }
            b = e;
        }
    }
    // row-length features: warp reduce, one atomic per warp
    for (int o = 16; o; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(0xffffffffu, mn, o));
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        sum += __shfl_xor_sync(0xffffffffu, sum, o);
        sq += __shfl_xor_sync(0xffffffffu, sq, o);
    }
    if (lane == 0) {
        atomicMin(&st->len_min, mn);
        atomicMax(&st->len_max, mx);
        atomicAdd(&st->len_sum, sum);
        atomicAdd(&st->len_sumsq, sq);
    }
    __syncthreads();
    for (int q = threadIdx.x; q < P * kMaxT; q += blockDim.x) {
        if (H_s[q]) atomicAdd(&st->H[0][0] + q, H_s[q]);
        if (F_s[q]) atomicAdd(&st->F[0][0] + q, F_s[q]);
    }
}

__global__ void __launch_bounds__(kThreads) stats_cols_kernel(const uint32_t *__restrict__ mask, int64_t n_cols,
                                                              int64_t S, int P, StatsDev *st) {
    extern __shared__ unsigned long long sh[];  // Un_s[P][32], Ut_s[P][32]
    unsigned long long *Un_s = sh, *Ut_s = sh + P * kMaxT;
    for (int q = threadIdx.x; q < 2 * P * kMaxT; q += blockDim.x) sh[q] = 0;
    __syncthreads();
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < n_cols; c += stride) {
        uint32_t m = mask[c];
        if (!m) continue;
        int p = (int)(c / S);
        int hb = 31 - __clz(m);
        for (int t = 0; t <= hb; t++) {
            if ((m >> t) & 1u) atomicAdd(&Un_s[p * kMaxT + t], 1ull);
            atomicAdd(&Ut_s[p * kMaxT + t], 1ull);
        }
    }
    __syncthreads();
    for (int q = threadIdx.x; q < P * kMaxT; q += blockDim.x) {
        if (Un_s[q]) atomicAdd(&st->Unat[0][0] + q, Un_s[q]);
        if (Ut_s[q]) atomicAdd(&st->Utop[0][0] + q, Ut_s[q]);
    }
}

int num_sms() {
    static int n = 0;
    if (!n) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        if (n <= 0) n = 148;
    }
    return n;
}

}  // namespace

cudaError_t launch_stats(const lf_csr &A, int P, StatsDev *d_stats, uint32_t *d_colmask, cudaStream_t s) {
    const int64_t S = A.n_cols > 0 ? (A.n_cols + P - 1) / P : 1;
    const size_t smem = 2 * (size_t)P * kMaxT * sizeof(unsigned long long);
    if (A.n_rows > 0) {
        int64_t want = (A.n_rows + kThreads - 1) / kThreads;
        int grid = (int)std::min<int64_t>(want, (int64_t)num_sms() * 8);
        stats_rows_kernel<<<grid, kThreads, smem, s>>>(A.row_ptr, A.col_ind, A.n_rows, S, P, d_stats, d_colmask);
    }
    if (A.n_cols > 0) {
        int64_t want = (A.n_cols + kThreads - 1) / kThreads;
        int grid = (int)std::min<int64_t>(want, (int64_t)num_sms() * 8);
        stats_cols_kernel<<<grid, kThreads, smem, s>>>(d_colmask, A.n_cols, S, P, d_stats);
    }
    return cudaGetLastError();
}

}  // namespace lf
