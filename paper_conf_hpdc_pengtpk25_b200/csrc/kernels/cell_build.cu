// cell_build.cu -- CSR -> CELL conversion on the GPU.
//
// The CELL layout (section 4; Fig. 4) is fixed
// by readings R1-R7: buckets partition-major / ascending width;
// inside a bucket ascending source row, a folded row's sub-rows consecutive,
// slots in CSR order; padding slots (-1, +0.0f); block-padding rows -1.  The
// result must equal the oracle's arrays bit for bit, so every placement is a
// deterministic, STABLE scan (no slot is claimed with an atomic):
//
//   a1  seg_kernel            segment starts of each row in partitions 1..P-1
//   a4  bucket_kernel<0>      per (tile of 256 rows, partition): bucket key
//                             t = min(ceil_log2 l, e_p), n_sub = ceil(l / 2^t),
//                             warp-stable ranks, per-tile per-key totals
//       tile_scan_kernel      exclusive scan over tiles per key (p, t)
//       (host)                bucket sizes -> padding -> bucket table
//       bucket_kernel<1>      CELL row position of every (row, partition):
//                             rowInd, and the CSR source of each CELL row
//   a5  slot_fill_kernel      warp per 256-slot chunk, lane-interleaved slots:
//                             colInd / val or padding
#include "../lf_internal.cuh"

namespace lf {

namespace {

constexpr int kThreads = kBuildTile;  // 256 rows per tile, one per thread
constexpr int kWarps = kThreads / 32;
constexpr int kNoKey = kMaxT;         // "empty segment"

__device__ __forceinline__ int64_t lower_bound_col(const int32_t *__restrict__ col, int64_t b, int64_t e,
                                                   int64_t v) {
    while (b < e) {
        int64_t m = (b + e) >> 1;
        if (col[m] < v) b = m + 1;
        else e = m;
    }
    return b;
}

__global__ void seg_kernel(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col, int64_t n_rows,
                           int64_t S, int P, int32_t *__restrict__ seg_rel) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_rows; i += stride) {
        const int64_t rb = row_ptr[i], re = row_ptr[i + 1];
        int64_t b = rb;
        for (int p = 1; p < P; p++) {
            b = lower_bound_col(col, b, re, (int64_t)p * S);
            seg_rel[i * (P - 1) + (p - 1)] = (int32_t)(b - rb);
        }
    }
}

// Segment [beg, end) of row i in partition p.
__device__ __forceinline__ void segment_of(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ seg_rel,
                                           int64_t i, int p, int P, int64_t &beg, int64_t &end) {
    const int64_t rb = row_ptr[i], re = row_ptr[i + 1];
    beg = (p == 0) ? rb : rb + seg_rel[i * (P - 1) + (p - 1)];
    end = (p == P - 1) ? re : rb + seg_rel[i * (P - 1) + p];
}

// PASS 0: count (tile totals + per-row CELL-row counts); PASS 1: place.
// A row folded into more than kThreadSubRows CELL rows has its sub-rows
// written by the whole warp (coalesced) instead of by its own thread.
#ifndef LF_THREAD_SUBROWS
#define LF_THREAD_SUBROWS 8  // measured (bucket_kernel<0>+<1> mean, us, c2/c3/c4): 32 -> 15.2/18.6/23.0, 8 -> 14.3/18.6/22.5, 4 -> 14.4/18.3/22.0, 1 -> 15.9/17.1/28.4
#endif
constexpr int kThreadSubRows = LF_THREAD_SUBROWS;
template <int PASS>
__global__ void __launch_bounds__(kThreads)
    bucket_kernel(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ seg_rel, int64_t n_rows, int P,
                  const __grid_constant__ WidthArg e_of_p, int n_tiles, long long *__restrict__ tile_cnt,
                  const long long *__restrict__ key_row_off, int32_t *__restrict__ row_cnt,
                  int32_t *__restrict__ row_ind, int32_t *__restrict__ row_tag, int64_t *__restrict__ src_pos,
                  int32_t *__restrict__ src_cnt, uint8_t *__restrict__ row_mode) {
    __shared__ long long warp_tot[kWarps][kMaxT];
    const int tile = blockIdx.x, p = blockIdx.y;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int64_t i = (int64_t)tile * kThreads + threadIdx.x;
    const int e = e_of_p.e[p];

    int64_t beg = 0, end = 0;
    if (i < n_rows) segment_of(row_ptr, seg_rel, i, p, P, beg, end);
    const int64_t l = end - beg;
    const int key = l > 0 ? min(ceil_log2_i64(l), e) : kNoKey;
    const int64_t n_sub = l > 0 ? (l + (int64_t(1) << key) - 1) >> key : 0;

    // warp-stable rank inside the key: rows of non-max buckets have n_sub = 1
    // (a count); the max bucket e needs a weighted (n_sub) prefix sum.
    const unsigned peers = __match_any_sync(0xffffffffu, key);
    const unsigned lt = (1u << lane) - 1u;
    long long v = (key == e) ? n_sub : 0, incl = v;
    for (int o = 1; o < 32; o <<= 1) {
        long long y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += y;
    }
    const long long top_total = __shfl_sync(0xffffffffu, incl, 31);
    const long long rank = (key == e) ? incl - v : (long long)__popc(peers & lt);
    if (threadIdx.x < kWarps * kMaxT) (&warp_tot[0][0])[threadIdx.x] = 0;
    __syncthreads();
    if (key != kNoKey && (peers & lt) == 0)  // key leader
        warp_tot[warp][key] = (key == e) ? top_total : (long long)__popc(peers);
    __syncthreads();
    if (threadIdx.x < kMaxT) {  // exclusive scan over warps, per key
        long long run = 0;
        for (int w = 0; w < kWarps; w++) {
            long long x = warp_tot[w][threadIdx.x];
            warp_tot[w][threadIdx.x] = run;
            run += x;
        }
        if (PASS == 0) tile_cnt[((int64_t)p * kMaxT + threadIdx.x) * n_tiles + tile] = run;
    }
    __syncthreads();

    if (PASS == 0) {
        if (P == 1) {  // every entry written: no memset
            if (i < n_rows) row_cnt[i] = (int32_t)n_sub;
        } else if (n_sub > 0) {
            atomicAdd(row_cnt + i, (int32_t)n_sub);
        }
        return;
    } else {
        int64_t pos = 0;
        int32_t tag = 0;
        if (key != kNoKey) {
            pos = key_row_off[p * kMaxT + key] + tile_cnt[((int64_t)p * kMaxT + key) * n_tiles + tile] +
                  warp_tot[warp][key] + rank;
            // (i << 3) | S << 2 | F << 1 | L  (cell_spmm.cu): S = the row is "whole":
            // this segment holds all of row i's CELL rows and one warp sums them
            // (single CELL row, or a run of <= kMaxRun rows in a wide bucket);
            // F / L mark the first / last sub-row and are added below
            const bool whole = row_cnt[i] == n_sub && key <= kPieceLog2 && (n_sub == 1 || (key >= 5 && n_sub <= kMaxRun));
            tag = (int32_t)((i << 3) | (whole ? 4 : 0));
            row_mode[i] = whole ? (n_sub == 1 ? kRowPlain : kRowRun) : kRowRed;
        } else if (P == 1 && i < n_rows) {
            row_mode[i] = kRowEmpty;  // (P > 1: pre-filled, another partition may own the row)
        }
        const int64_t W = int64_t(1) << (key == kNoKey ? 0 : key);
        if (n_sub <= kThreadSubRows) {
            for (int64_t s = 0; s < n_sub; s++) {
                row_ind[pos + s] = (int32_t)i;
                row_tag[pos + s] = tag | (s == 0 ? 2 : 0) | (s == n_sub - 1 ? 1 : 0);
                src_pos[pos + s] = beg + s * W;
                src_cnt[pos + s] = (int32_t)min(W, l - s * W);
            }
        }
        // long folded rows: the warp writes their sub-rows together
        unsigned long_lanes = __ballot_sync(0xffffffffu, n_sub > kThreadSubRows);
        while (long_lanes) {
            const int src = __ffs(long_lanes) - 1;
            long_lanes &= long_lanes - 1;
            const int64_t sp = __shfl_sync(0xffffffffu, pos, src);
            const int64_t sb = __shfl_sync(0xffffffffu, beg, src);
            const int64_t sl = __shfl_sync(0xffffffffu, l, src);
            const int64_t sn = __shfl_sync(0xffffffffu, n_sub, src);
            const int64_t sW = __shfl_sync(0xffffffffu, W, src);
            const int32_t stag = __shfl_sync(0xffffffffu, tag, src);
            const int64_t si = __shfl_sync(0xffffffffu, i, src);
            for (int64_t s = lane; s < sn; s += 32) {
                row_ind[sp + s] = (int32_t)si;
                row_tag[sp + s] = stag | (s == 0 ? 2 : 0) | (s == sn - 1 ? 1 : 0);
                src_pos[sp + s] = sb + s * sW;
                src_cnt[sp + s] = (int32_t)min(sW, sl - s * sW);
            }
        }
    }
}

// exclusive scan over n_tiles entries of each key (p, t); one block per key
__global__ void __launch_bounds__(1024) tile_scan_kernel(long long *__restrict__ tile_cnt, int n_tiles,
                                                         long long *__restrict__ key_total) {
    __shared__ long long wsum[32];
    __shared__ long long carry;
    long long *x = tile_cnt + (int64_t)blockIdx.x * n_tiles;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (int base = 0; base < n_tiles; base += 1024) {
        const int q = base + threadIdx.x;
        const long long v = q < n_tiles ? x[q] : 0;
        long long incl = v;
        for (int o = 1; o < 32; o <<= 1) {
            long long y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
        }
        if (lane == 31) wsum[warp] = incl;
        __syncthreads();
        if (warp == 0) {
            long long w = wsum[lane], wi = w;
            for (int o = 1; o < 32; o <<= 1) {
                long long y = __shfl_up_sync(0xffffffffu, wi, o);
                if (lane >= o) wi += y;
            }
            wsum[lane] = wi - w;  // exclusive prefix of warp sums
        }
        __syncthreads();
        const long long c0 = carry;
        if (q < n_tiles) x[q] = c0 + wsum[warp] + incl - v;
        __syncthreads();
        if (threadIdx.x == 1023) carry = c0 + wsum[warp] + incl;
        __syncthreads();
    }
    if (threadIdx.x == 0) key_total[blockIdx.x] = carry;
}

// one block per bucket: its block-padding rows, and (block 0) the counters
__global__ void pad_init_kernel(const BucketDev *__restrict__ bk, int nb, int32_t *__restrict__ row_ind,
                                int32_t *__restrict__ row_tag, int32_t *__restrict__ src_cnt,
                                int64_t *__restrict__ src_pos, unsigned long long *__restrict__ ctr, int n_ctr) {
    if (blockIdx.x == 0)
        for (int q = threadIdx.x; q < n_ctr; q += blockDim.x) ctr[q] = 0;
    if ((int)blockIdx.x >= nb) return;
    const BucketDev b = bk[blockIdx.x];
    for (int64_t r = b.row_off + b.n_real_rows + threadIdx.x; r < b.row_off + b.n_rows_pad; r += blockDim.x) {
        row_ind[r] = -1;
        row_tag[r] = -1;
        src_cnt[r] = 0;
        src_pos[r] = 0;  // never dereferenced (count 0), but defined (initcheck)
    }
}

constexpr int kSlotThreads = 256;
constexpr int kMaxSmemBuckets = 2048;
#ifndef LF_SLOTS_PER_LANE
#define LF_SLOTS_PER_LANE 8  // measured (us, c2/c3/c4): 4 -> 71/207/585, 8 -> 70/199/525, 16 slower
#endif
constexpr int kSlotsPerLane = LF_SLOTS_PER_LANE;    // consecutive slots per lane: 16-byte stores
constexpr int kSlotsPerWarp = 32 * kSlotsPerLane;   // a warp's chunk

// A warp fills 32 * kSlotsPerLane consecutive slots per chunk, lane l taking
// slots l, l + 32, ... (coalesced CSR reads and C-ABI array writes).
// The bucket of the chunk is found once (warp-uniform binary search over the
// bucket slot offsets in shared memory); a chunk that straddles buckets
// falls back to a per-slot search.  Slot s of bucket b is position
// w = (s - soff) mod W of CELL row r = roff + (s - soff) / W; it copies
// colInd / val from CSR position src_pos[r] + w when w < src_cnt[r]
// (0 for block-padding rows), else the padding (-1, +0.0f).
__device__ __forceinline__ int bucket_of(const int64_t *soff, int nb, int64_t s) {
    int lo = 0, hi = nb - 1;  // last bucket with soff <= s
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (soff[mid] <= s) lo = mid;
        else hi = mid - 1;
    }
    return lo;
}

__global__ void __launch_bounds__(kSlotThreads)
    slot_fill_kernel(const int32_t *__restrict__ col, const float *__restrict__ val,
                     const BucketDev *__restrict__ bk, int nb, int64_t n_slots, const int64_t *__restrict__ src_pos,
                     const int32_t *__restrict__ src_cnt, int32_t *__restrict__ col_out,
                     float *__restrict__ val_out) {
    __shared__ int64_t soff[kMaxSmemBuckets];
    __shared__ int64_t roff[kMaxSmemBuckets];
    __shared__ int32_t tt[kMaxSmemBuckets];
    for (int q = threadIdx.x; q < nb; q += blockDim.x) {
        soff[q] = bk[q].slot_off;
        roff[q] = bk[q].row_off;
        tt[q] = bk[q].t;
    }
    __syncthreads();
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t ch = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; ch * kSlotsPerWarp < n_slots; ch += nw) {
        const int64_t c0 = ch * kSlotsPerWarp;
        const int bu = bucket_of(soff, nb, c0);  // uniform
        const bool one = bu + 1 >= nb || soff[bu + 1] >= c0 + kSlotsPerWarp;
#ifndef LF_SLOT_INTERLEAVE
#define LF_SLOT_INTERLEAVE 1  // slot k of lane l is c0 + 32 k + l (coalesced loads, 4-byte coalesced stores);
                              // 0: 8 consecutive slots per lane, 16-byte stores (c2 69.9 -> 56.4 us with 1)
#endif
        const int64_t s0 = LF_SLOT_INTERLEAVE ? c0 + lane : c0 + lane * kSlotsPerLane;
        constexpr int kStep = LF_SLOT_INTERLEAVE ? 32 : 1;
        int32_t c[kSlotsPerLane];
        float v[kSlotsPerLane];
        int64_t pos[kSlotsPerLane];
        int32_t cnt[kSlotsPerLane], w[kSlotsPerLane];
#pragma unroll
        for (int k = 0; k < kSlotsPerLane; k++) {
            const int64_t s = s0 + k * kStep;
            cnt[k] = 0;
            w[k] = 1;
            pos[k] = 0;
            if (s < n_slots) {
                const int b = one ? bu : bucket_of(soff, nb, s);
                const int t = tt[b];
                const int64_t rel = s - soff[b];
                const int64_t r = roff[b] + (rel >> t);
                w[k] = (int32_t)(rel & ((int64_t(1) << t) - 1));
                cnt[k] = __ldg(src_cnt + r);
                pos[k] = __ldg(src_pos + r);
            }
        }
#pragma unroll
        for (int k = 0; k < kSlotsPerLane; k++) {
            const bool real = w[k] < cnt[k];
            c[k] = real ? __ldg(col + pos[k] + w[k]) : -1;
            v[k] = real ? __ldg(val + pos[k] + w[k]) : 0.0f;
        }
        if (LF_SLOT_INTERLEAVE) {
#pragma unroll
            for (int k = 0; k < kSlotsPerLane; k++)
                if (s0 + k * kStep < n_slots) {
                    __stcs(col_out + s0 + k * kStep, c[k]);
                    __stcs(val_out + s0 + k * kStep, v[k]);
                }
        } else if (s0 + kSlotsPerLane <= n_slots) {
#pragma unroll
            for (int k = 0; k < kSlotsPerLane; k += 4) {
                __stcs(reinterpret_cast<int4 *>(col_out + s0 + k), make_int4(c[k], c[k + 1], c[k + 2], c[k + 3]));
                __stcs(reinterpret_cast<float4 *>(val_out + s0 + k), make_float4(v[k], v[k + 1], v[k + 2], v[k + 3]));
            }
        } else {
#pragma unroll
            for (int k = 0; k < kSlotsPerLane; k++)
                if (s0 + k < n_slots) {
                    __stcs(col_out + s0 + k, c[k]);
                    __stcs(val_out + s0 + k, v[k]);
                }
        }
    }
}

// run_bound[x] for every wide task x (0..n): offset to the first task >= x
// that starts a run (F), is a padding row, or belongs to a row written with
// atomics (!S); n counts as a bound.  A whole run (<= kMaxRun <= 32 CELL
// rows) never straddles two work claims whose ends are aligned this way.
// One warp per 32 positions, over a 64-task window of boundary flags.
__device__ __forceinline__ bool is_bound(const BucketDev *__restrict__ bk, int nb, int64_t n,
                                         const int32_t *__restrict__ tag, int64_t p) {
    if (p >= n) return true;
    int lo = 0, hi = nb - 1;  // bucket of task p
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (bk[mid].task_off <= p) lo = mid;
        else hi = mid - 1;
    }
    const int32_t tg = tag[bk[lo].row_off + ((p - bk[lo].task_off) >> bk[lo].piece_log2)];
    return tg < 0 || (tg & 2) || !(tg & 4);
}

__global__ void run_bounds_kernel(const BucketDev *__restrict__ bk, int nb, int64_t n, const int32_t *__restrict__ tag,
                                  uint8_t *__restrict__ out, int64_t n_out) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w * 32 < n_out; w += nw) {
        const int64_t x0 = w * 32;
        const unsigned m1 = __ballot_sync(0xffffffffu, is_bound(bk, nb, n, tag, x0 + lane));
        const unsigned m2 = __ballot_sync(0xffffffffu, is_bound(bk, nb, n, tag, x0 + 32 + lane));
        const unsigned long long m = ((unsigned long long)m2 << 32 | m1) >> lane;  // bit 0 = position x0 + lane
        if (x0 + lane < n_out) out[x0 + lane] = (uint8_t)(m ? min(__ffsll((long long)m) - 1, 32) : 32);
    }
}

__global__ void validate_kernel(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col, int64_t n_rows,
                                int64_t n_cols, int *flag) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_rows; i += stride) {
        const int64_t rb = row_ptr[i], re = row_ptr[i + 1];
        if (re < rb) { atomicOr(flag, 2); continue; }
        for (int64_t q = rb; q < re; q++) {
            const int32_t c = col[q];
            if (c < 0 || c >= n_cols) atomicOr(flag, 2);
            if (q > rb && col[q - 1] > c) atomicOr(flag, 1);
        }
    }
}

int grid_for(int64_t n, int threads) {
    int64_t g = (n + threads - 1) / threads;
    return (int)std::max<int64_t>(1, std::min<int64_t>(g, (int64_t)sm_count() * 32));
}

}  // namespace

cudaError_t launch_seg(const lf_csr &A, int P, int32_t *seg_rel, cudaStream_t s) {
    if (P <= 1 || A.n_rows == 0) return cudaSuccess;
    const int64_t S = (A.n_cols + P - 1) / P;
    seg_kernel<<<grid_for(A.n_rows, 256), 256, 0, s>>>(A.row_ptr, A.col_ind, A.n_rows, S, P, seg_rel);
    return cudaGetLastError();
}

cudaError_t launch_bucket_count(const lf_csr &A, int P, const WidthArg &e, const BuildScratch &sc, int32_t *row_cnt,
                                cudaStream_t s) {
    if (A.n_rows == 0) return cudaSuccess;
    dim3 grid(sc.n_tiles, P);
    bucket_kernel<0><<<grid, kThreads, 0, s>>>(A.row_ptr, sc.seg_rel, A.n_rows, P, e, sc.n_tiles, sc.tile_cnt,
                                                nullptr, row_cnt, nullptr, nullptr, nullptr, nullptr, nullptr);
    return cudaGetLastError();
}

cudaError_t launch_tile_scan(int P, const BuildScratch &sc, cudaStream_t s) {
    tile_scan_kernel<<<P * kMaxT, 1024, 0, s>>>(sc.tile_cnt, sc.n_tiles, sc.key_total);
    return cudaGetLastError();
}

cudaError_t launch_pad_init(const BucketDev *bk, int nb, int32_t *row_ind, int32_t *row_tag, int32_t *src_cnt,
                            int64_t *src_pos, unsigned long long *ctr, int n_ctr, cudaStream_t s) {
    pad_init_kernel<<<std::max(nb, 1), 256, 0, s>>>(bk, nb, row_ind, row_tag, src_cnt, src_pos, ctr, n_ctr);
    return cudaGetLastError();
}

cudaError_t launch_bucket_place(const lf_csr &A, int P, const WidthArg &e, const BuildScratch &sc,
                                const int32_t *row_cnt, int32_t *row_ind, int32_t *row_tag, uint8_t *row_mode,
                                cudaStream_t s) {
    if (A.n_rows == 0) return cudaSuccess;
    dim3 grid(sc.n_tiles, P);
    bucket_kernel<1><<<grid, kThreads, 0, s>>>(A.row_ptr, sc.seg_rel, A.n_rows, P, e, sc.n_tiles, sc.tile_cnt,
                                                sc.key_row_off, const_cast<int32_t *>(row_cnt), row_ind, row_tag,
                                                sc.src_pos, sc.src_cnt, row_mode);
    return cudaGetLastError();
}

cudaError_t launch_slot_fill(const lf_csr &A, const BucketDev *d_buckets, int nb, int64_t n_slots,
                             const BuildScratch &sc, int32_t *col_out, float *val_out, cudaStream_t s) {
    if (n_slots == 0) return cudaSuccess;
    if (nb > kMaxSmemBuckets) return cudaErrorInvalidValue;
    static_assert(kSlotsPerLane % 4 == 0, "vector stores");
    slot_fill_kernel<<<grid_for((n_slots + kSlotsPerLane - 1) / kSlotsPerLane, kSlotThreads), kSlotThreads, 0, s>>>(
        A.col_ind, A.val, d_buckets, nb, n_slots, sc.src_pos, sc.src_cnt, col_out, val_out);
    return cudaGetLastError();
}

cudaError_t launch_run_bounds(const BucketDev *bk_w, int nb_w, int64_t n_tasks_w, const int32_t *row_tag,
                              uint8_t *run_bound, cudaStream_t s) {
    const int64_t n_out = n_tasks_w + 1;
    if (nb_w == 0) return cudaMemsetAsync(run_bound, 0, (size_t)n_out, s);
    run_bounds_kernel<<<grid_for(n_out, 256), 256, 0, s>>>(bk_w, nb_w, n_tasks_w, row_tag, run_bound, n_out);
    return cudaGetLastError();
}

cudaError_t launch_validate(const lf_csr &A, int *d_flag, cudaStream_t s) {
    if (A.n_rows == 0) return cudaSuccess;
    validate_kernel<<<grid_for(A.n_rows, 256), 256, 0, s>>>(A.row_ptr, A.col_ind, A.n_rows, A.n_cols, d_flag);
    return cudaGetLastError();
}

}  // namespace lf
