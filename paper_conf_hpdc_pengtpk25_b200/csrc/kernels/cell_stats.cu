// cell_stats.cu -- configure statistics on the GPU.
//
// For every partition p and natural bucket t = ceil_log2(l) of every
// non-empty row segment (reading R1) the host needs
//   H[p][t]  segment count,  F[p][t] = sum_{t0 >= t} ceil(l / 2^t)  (fold rows),
//   Unat[p][t], Utop[p][t]   the |set(Ind)| terms of eq. 7
// plus the Table 2 row-length statistics.  Three passes:
//   stats_rows_kernel   one thread per row: segments, H, F (warp-aggregated
//                       with REDUX), features; writes t0 of every segment
//   stats_mark_kernel   nnz-balanced: column c of segment (i,p) sets bit t0 of
//                       a per-column mask M[c] (partition of c is c / S)
//   stats_cols_kernel   one thread per column: Unat[p][t] = #{c : bit t},
//                       Utop[p][t] = #{c : highest bit >= t} (warp-aggregated)
#include "../lf_internal.cuh"

namespace lf {

namespace {

constexpr int kThreads = 256;
constexpr int kMarkPerThread = 16;
constexpr int kMarkTile = kThreads * kMarkPerThread;
constexpr unsigned kFull = 0xffffffffu;
constexpr uint8_t kEmpty = 0xFF;

__device__ __forceinline__ int64_t lower_bound_col(const int32_t *__restrict__ col, int64_t b, int64_t e,
                                                   int64_t v) {
    while (b < e) {
        int64_t m = (b + e) >> 1;
        if (col[m] < v) b = m + 1;
        else e = m;
    }
    return b;
}

// warp sum of a non-negative value < 2^31 into a 64-bit result (two REDUX)
__device__ __forceinline__ unsigned long long warp_sum_u31(unsigned v) {
    unsigned lo = __reduce_add_sync(kFull, v & 0xFFFFu);
    unsigned hi = __reduce_add_sync(kFull, v >> 16);
    return ((unsigned long long)hi << 16) + lo;
}

__global__ void __launch_bounds__(kThreads) stats_rows_kernel(const int64_t *__restrict__ row_ptr,
                                                              const int32_t *__restrict__ col, int64_t n_rows,
                                                              int64_t S, int P, StatsDev *st,
                                                              uint8_t *__restrict__ t0seg) {
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
            const int64_t e = (p == P - 1) ? re : lower_bound_col(col, b, re, (int64_t)(p + 1) * S);
            const int64_t l = e - b;
            const int t0 = l > 0 ? ceil_log2_i64(l) : kMaxT;
            if (active) t0seg[i * P + p] = l > 0 ? (uint8_t)t0 : kEmpty;
            // H: one shared atomic per distinct t0 in the warp
            const unsigned peers = __match_any_sync(kFull, t0);
            if (t0 < kMaxT && (peers & ((1u << lane) - 1u)) == 0)
                atomicAdd(&H_s[p * kMaxT + t0], (unsigned long long)__popc(peers));
            // F[t] for t <= t0 (REDUX per level up to the warp's largest t0)
            const int tmax = __reduce_max_sync(kFull, l > 0 ? (unsigned)t0 : 0u);
            const bool any = __any_sync(kFull, l > 0);
            if (any) {
                for (int t = 0; t <= tmax; t++) {
                    unsigned v = (l > 0 && t <= t0) ? (unsigned)((l + (int64_t(1) << t) - 1) >> t) : 0u;
                    unsigned long long s = warp_sum_u31(v);
                    if (lane == 0 && s) atomicAdd(&F_s[p * kMaxT + t], s);
                }
            }
            b = e;
        }
    }
    for (int o = 16; o; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(kFull, mn, o));
        mx = max(mx, __shfl_xor_sync(kFull, mx, o));
        sum += __shfl_xor_sync(kFull, sum, o);
        sq += __shfl_xor_sync(kFull, sq, o);
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

// nnz-balanced column marking.  Positions q of tile [q0, q0 + kMarkTile) are
// mapped to their row by a binary search in row_ptr restricted to the tile's
// row range (found once per block).
__global__ void __launch_bounds__(kThreads) stats_mark_kernel(const int64_t *__restrict__ row_ptr,
                                                              const int32_t *__restrict__ col, int64_t n_rows,
                                                              int64_t S, int P,
                                                              const uint8_t *__restrict__ t0seg,
                                                              uint32_t *__restrict__ mask) {
    __shared__ int64_t rng[2];
    const int64_t base = row_ptr[0];
    const int64_t nnz = row_ptr[n_rows] - base;
    for (int64_t q0 = (int64_t)blockIdx.x * kMarkTile; q0 < nnz; q0 += (int64_t)gridDim.x * kMarkTile) {
        if (threadIdx.x < 2) {
            // last row r with row_ptr[r] - base <= target
            const int64_t target = threadIdx.x == 0 ? q0 : min(q0 + kMarkTile, nnz) - 1;
            int64_t lo = 0, hi = n_rows - 1;
            while (lo < hi) {
                int64_t m = (lo + hi + 1) >> 1;
                if (row_ptr[m] - base <= target) lo = m;
                else hi = m - 1;
            }
            rng[threadIdx.x] = lo;
        }
        __syncthreads();
        const int64_t rlo = rng[0], rhi = rng[1];
#pragma unroll 4
        for (int k = 0; k < kMarkPerThread; k++) {
            const int64_t q = q0 + k * kThreads + threadIdx.x;
            if (q >= nnz) break;
            int64_t lo = rlo, hi = rhi;
            while (lo < hi) {
                int64_t m = (lo + hi + 1) >> 1;
                if (row_ptr[m] - base <= q) lo = m;
                else hi = m - 1;
            }
            const int32_t c = col[base + q];
            const int p = P == 1 ? 0 : (int)(c / S);
            const uint32_t bit = 1u << t0seg[lo * P + p];
            if (!(__ldcg(mask + c) & bit)) atomicOr(mask + c, bit);
        }
        __syncthreads();
    }
}

__global__ void __launch_bounds__(kThreads) stats_cols_kernel(const uint32_t *__restrict__ mask, int64_t n_cols,
                                                              int64_t S, int P, StatsDev *st) {
    extern __shared__ unsigned long long sh[];  // Un_s[P][32], Ut_s[P][32]
    unsigned long long *Un_s = sh, *Ut_s = sh + P * kMaxT;
    for (int q = threadIdx.x; q < 2 * P * kMaxT; q += blockDim.x) sh[q] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n_cols; base += stride) {
        const int64_t c = base + threadIdx.x;
        const uint32_t m = c < n_cols ? mask[c] : 0u;
        const int p = c < n_cols ? (int)(c / S) : -1;
        const int hb = m ? 31 - __clz(m) : -1;
        // columns of one warp may straddle a partition boundary: group by p
        unsigned todo = __ballot_sync(kFull, m != 0);
        while (todo) {
            const int pp = __shfl_sync(kFull, p, __ffs(todo) - 1);
            const bool mine = m != 0 && p == pp;
            todo &= ~__ballot_sync(kFull, mine);
            const int tmax = __reduce_max_sync(kFull, mine ? (unsigned)hb : 0u);
            for (int t = 0; t <= tmax; t++) {
                const unsigned un = __reduce_add_sync(kFull, mine && ((m >> t) & 1u));
                const unsigned ut = __reduce_add_sync(kFull, mine && hb >= t);
                if (lane == 0) {
                    if (un) atomicAdd(&Un_s[pp * kMaxT + t], (unsigned long long)un);
                    if (ut) atomicAdd(&Ut_s[pp * kMaxT + t], (unsigned long long)ut);
                }
            }
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

cudaError_t launch_stats(const lf_csr &A, int P, StatsDev *d_stats, uint32_t *d_colmask, uint8_t *d_t0seg,
                         cudaStream_t s) {
    const int64_t S = A.n_cols > 0 ? (A.n_cols + P - 1) / P : 1;
    const size_t smem = 2 * (size_t)P * kMaxT * sizeof(unsigned long long);
    if (A.n_rows > 0) {
        int64_t want = (A.n_rows + kThreads - 1) / kThreads;
        int grid = (int)std::min<int64_t>(want, (int64_t)num_sms() * 8);
        stats_rows_kernel<<<grid, kThreads, smem, s>>>(A.row_ptr, A.col_ind, A.n_rows, S, P, d_stats, d_t0seg);
        if (A.nnz > 0) {
            int64_t tiles = (A.nnz + kMarkTile - 1) / kMarkTile;
            int g2 = (int)std::min<int64_t>(tiles, (int64_t)num_sms() * 8);
            stats_mark_kernel<<<g2, kThreads, 0, s>>>(A.row_ptr, A.col_ind, A.n_rows, S, P, d_t0seg, d_colmask);
        }
    }
    if (A.n_cols > 0) {
        int64_t want = (A.n_cols + kThreads - 1) / kThreads;
        int grid = (int)std::min<int64_t>(want, (int64_t)num_sms() * 8);
        stats_cols_kernel<<<grid, kThreads, smem, s>>>(d_colmask, A.n_cols, S, P, d_stats);
    }
    return cudaGetLastError();
}

}  // namespace lf
