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

// nnz-balanced column marking.  Every lane owns kMarkPerThread consecutive
// positions: one binary search in row_ptr finds the row of its first
// position, then rows advance as positions cross row_ptr boundaries.
// Power-law inputs send a large share of all nonzeros to a few hot columns
// whose mask words share L2 lines, so a per-block direct-mapped filter in
// shared memory ((col << 32) | bits already set globally, one 64-bit word per
// slot, updated with whole-word stores so a (col, bits) pair is always
// consistent) drops repeated (col, bit) pairs before they reach L2.
constexpr int kFilter = 4096;

__global__ void __launch_bounds__(kThreads) stats_mark_kernel(const int64_t *__restrict__ row_ptr,
                                                              const int32_t *__restrict__ col, int64_t n_rows,
                                                              int64_t S, int P,
                                                              const uint8_t *__restrict__ t0seg,
                                                              uint32_t *__restrict__ mask) {
    __shared__ unsigned long long filt[kFilter];
    for (int q = threadIdx.x; q < kFilter; q += blockDim.x) filt[q] = ~0ull;  // col field 0xFFFFFFFF: empty
    __syncthreads();
    const int64_t base = row_ptr[0];
    const int64_t nnz = row_ptr[n_rows] - base;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x * kMarkPerThread;
    for (int64_t q0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * kMarkPerThread; q0 < nnz; q0 += stride) {
        // row of position q0: last r with row_ptr[r] - base <= q0
        int64_t lo = 0, hi = n_rows - 1;
        while (lo < hi) {
            const int64_t m = (lo + hi + 1) >> 1;
            if (__ldg(row_ptr + m) - base <= q0) lo = m;
            else hi = m - 1;
        }
        int64_t r = lo;
        int64_t rend = __ldg(row_ptr + r + 1) - base;
        int32_t c[kMarkPerThread];
        uint32_t bit[kMarkPerThread];
#pragma unroll
        for (int k = 0; k < kMarkPerThread; k++) {
            const int64_t q = q0 + k;
            c[k] = -1;
            bit[k] = 0;
            if (q < nnz) {
                while (q >= rend) rend = __ldg(row_ptr + (++r) + 1) - base;
                c[k] = __ldg(col + base + q);
                const int p = P == 1 ? 0 : (int)(c[k] / S);
                bit[k] = 1u << __ldg(t0seg + r * P + p);
            }
        }
#pragma unroll
        for (int k = 0; k < kMarkPerThread; k++) {
            if (c[k] < 0) continue;
            const int slot = c[k] & (kFilter - 1);
            const unsigned long long f = filt[slot];
            const bool same = (uint32_t)(f >> 32) == (uint32_t)c[k];
            if (same && ((uint32_t)f & bit[k])) continue;
            atomicOr(mask + c[k], bit[k]);
            filt[slot] = ((unsigned long long)(uint32_t)c[k] << 32) | (same ? ((uint32_t)f | bit[k]) : bit[k]);
        }
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
            int g2 = (int)std::min<int64_t>(tiles, (int64_t)num_sms() * 16);
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
