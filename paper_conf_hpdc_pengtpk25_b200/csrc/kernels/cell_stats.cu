// cell_stats.cu -- configure statistics on the GPU.
//
// For every partition p and natural bucket t = ceil_log2(l) of every
// non-empty row segment (reading R1) the host needs
//   H[p][t]  segment count,  F[p][t] = sum_{t0 >= t} ceil(l / 2^t)  (fold rows),
//   Unat[p][t], Utop[p][t]   the |set(Ind)| terms of eq. 7
// plus the Table 2 row-length statistics.  Three passes:
//   stats_rows_kernel   one thread per row: segments, H, F (warp-aggregated),
//                       features; t0 of every segment -> t0seg; merge-path
//                       tiles of the marking pass
//   stats_mark_kernel   nnz-balanced tiles: every nonzero sets bit t0 of its
//                       segment in the per-column mask M[c] (partition of c
//                       is c / S); tiles of one natural bucket merge their
//                       (column, bits) pairs in a shared-memory filter first
//   stats_cols_kernel   one thread per mask slot: Unat[p][t] = #{c : bit t},
//                       Utop[p][t] = #{c : highest bit >= t} (bit transpose)
// and, for the grouped / windowed SpMM paths' decision, the group samples
// (group_sample_warp: distinct columns of 4-row groups, B-row windows of
// 128-row groups), taken by extra blocks of stats_rows_kernel or, on the
// features-first path, of features_kernel; features_kernel reads the row
// lengths alone when the statistics pass is not run speculatively (lf_api.cu).
#include "../lf_internal.cuh"

namespace lf {

namespace {

constexpr int kThreads = 256;
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

// Block reduction of the four row-length statistics, then one set of 64-bit
// atomics per block (per-warp atomics on the same four words serialise).
__device__ __forceinline__ void block_len_stats(unsigned long long mn, unsigned long long mx, unsigned long long sum,
                                                unsigned long long sq, StatsDev *st) {
    __shared__ unsigned long long red[4][kThreads / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int o = 16; o; o >>= 1) {
        mn = min(mn, __shfl_xor_sync(kFull, mn, o));
        mx = max(mx, __shfl_xor_sync(kFull, mx, o));
        sum += __shfl_xor_sync(kFull, sum, o);
        sq += __shfl_xor_sync(kFull, sq, o);
    }
    if (lane == 0) {
        red[0][warp] = mn;
        red[1][warp] = mx;
        red[2][warp] = sum;
        red[3][warp] = sq;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < (int)(blockDim.x >> 5); w++) {
            mn = min(mn, red[0][w]);
            mx = max(mx, red[1][w]);
            sum += red[2][w];
            sq += red[3][w];
        }
        atomicMin(&st->len_min, mn);
        atomicMax(&st->len_max, mx);
        atomicAdd(&st->len_sum, sum);
        atomicAdd(&st->len_sumsq, sq);
    }
}

// Grouped-path heuristic (cell_spmm.cu "grouped path"): on kGroupSamples
// groups of kGroupRows consecutive rows spread evenly over A (rows of at most
// 32 nonzeros; a group with a longer row is skipped), the number of DISTINCT
// columns of the group and its nonzeros, summed.  Their ratio says how many
// B-row gathers merging the group's columns saves.  A warp per group, the
// distinct columns counted in a per-warp shared-memory hash set.
constexpr int kGroupSamples = 2048;
__device__ __forceinline__ void group_sample_warp(const int64_t *__restrict__ row_ptr,
                                                  const int32_t *__restrict__ col, int64_t n_rows, StatsDev *st,
                                                  int64_t smp, int32_t *hs_w) {
    const int lane = threadIdx.x & 31;
    for (int q = lane; q < 256; q += 32) hs_w[q] = -1;
    __syncwarp();
    if (smp >= kGroupSamples) return;
    // tcgen05 windowed path (cell_spmm_tc.cu): the B-row window of 128
    // consecutive rows = [min first column, max last column]; rows longer than
    // 32 make the sample ineligible (the path needs every W <= 32)
    {
        const int64_t n_wg = n_rows / 128;
        if (n_wg > 0) {
            const int64_t i0 = (smp * n_wg / kGroupSamples) * 128;
            const int64_t base0 = row_ptr[0];
            int mn = INT32_MAX, mx = -1;
            bool ok = true;
            for (int r = lane; r < 128; r += 32) {
                const int64_t b = row_ptr[i0 + r] - base0, e = row_ptr[i0 + r + 1] - base0;
                ok = ok && e - b <= 32;
                if (e > b) {
                    mn = min(mn, col[base0 + b]);
                    mx = max(mx, col[base0 + e - 1]);
                }
            }
            ok = __all_sync(kFull, ok);
            mn = __reduce_min_sync(kFull, mn);
            mx = __reduce_max_sync(kFull, mx);
            if (lane == 0 && ok && mx >= 0) {
                const unsigned long long span = (unsigned long long)(mx - mn + 1);
                atomicAdd(&st->win_span, span);
                atomicAdd(&st->win_cnt, 1ull);
                if (span > 256) atomicAdd(&st->win_over, 1ull);
            }
        }
    }
    const int64_t n_groups = n_rows / kGroupRows;
    if (n_groups == 0) return;
    const int64_t i0 = (smp * n_groups / kGroupSamples) * kGroupRows;
    const int64_t base = row_ptr[0];
    int64_t b[kGroupRows], l[kGroupRows];
    bool ok = true;
#pragma unroll
    for (int r = 0; r < kGroupRows; r++) {
        b[r] = row_ptr[i0 + r] - base;
        l[r] = row_ptr[i0 + r + 1] - base - b[r];
        ok = ok && l[r] <= 32;
    }
    if (!ok) return;
    const int32_t *colb = col + base;
    unsigned n_u = 0, n_nz = 0;
#pragma unroll
    for (int r = 0; r < kGroupRows; r++) {
        const int32_t c = lane < l[r] ? colb[b[r] + lane] : -1;
        bool need = c >= 0, ins = false;
        int h = (int)(((uint32_t)c * 0x9E3779B1u) >> 24);
        while (__any_sync(kFull, need)) {
            if (need) {
                const int prev = atomicCAS(&hs_w[h], -1, c);
                if (prev == -1) ins = true;
                if (prev == -1 || prev == c) need = false;
                else h = (h + 1) & 255;
            }
        }
        n_u += __popc(__ballot_sync(kFull, ins));
        n_nz += (unsigned)l[r];
    }
    if (lane == 0) {
        atomicAdd(&st->grp_union, (unsigned long long)n_u);
        atomicAdd(&st->grp_nnz, (unsigned long long)n_nz);
    }
}

// Pass 1 -- one thread per row: segments of the row in every partition, their
// natural bucket t0 (written to t0seg[i*P+p]), the H / F histograms
// (warp-aggregated: __match_any_sync for H, REDUX for F) and the Table 2
// row-length statistics.
#ifndef LF_MARK_TILE
#define LF_MARK_TILE 4096  // items (row ends + nonzeros) per block of the marking pass
#endif
constexpr int kMarkTile = LF_MARK_TILE;
#ifndef LF_MARK_MIN_BLOCKS
#define LF_MARK_MIN_BLOCKS 4  // resident marking blocks per SM (64 registers)
#endif

__global__ void __launch_bounds__(kThreads) stats_rows_kernel(const int64_t *__restrict__ row_ptr,
                                                              const int32_t *__restrict__ col, int64_t n_rows,
                                                              int64_t S, int P, StatsDev *st,
                                                              uint8_t *__restrict__ t0seg,
                                                              int64_t *__restrict__ tile_row,
                                                              int64_t *__restrict__ tile_pos, int rows_grid) {
    if ((int)blockIdx.x >= rows_grid) {
        // the blocks after the row blocks take the grouped / windowed path samples
        // (group_sample_warp): independent of the row pass, so they run beside it
        __shared__ int32_t hs[8][256];
        const int w = threadIdx.x >> 5;
        group_sample_warp(row_ptr, col, n_rows, st, (int64_t)(blockIdx.x - rows_grid) * 8 + w, hs[w]);
        return;
    }
    extern __shared__ unsigned long long sh[];  // H_s[P][32], F_s[P][32]
    unsigned long long *H_s = sh, *F_s = sh + P * kMaxT;
    for (int q = threadIdx.x; q < 2 * P * kMaxT; q += blockDim.x) sh[q] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    unsigned long long mn = ~0ull, mx = 0, sum = 0, sq = 0;
    // P = 1: lane t keeps H[t] / F[t] of its warp in registers (a 64-bit
    // shared-memory atomicAdd is a CAS loop: per row batch it was a quarter
    // of the kernel's instructions); added to the block's table once
    unsigned long long accH = 0, accF = 0;
    const int64_t stride = (int64_t)rows_grid * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n_rows; base += stride) {
        const int64_t i = base + threadIdx.x;
        const bool active = i < n_rows;
        int64_t rb = 0, re = 0;
        if (active) {
            rb = row_ptr[i];
            re = row_ptr[i + 1];
            const unsigned long long len = (unsigned long long)(re - rb);
            // merge-path tiles over items = (row ends, nonzeros): row i owns items
            // [rb + i, re + i + 1); tile T starts at item T * kMarkTile, inside
            // row tile_row[T] at position tile_pos[T] (relative to row_ptr[0])
            const int64_t base = row_ptr[0];
            const int64_t b_item = rb - base + i, e_item = re - base + i + 1;
            for (int64_t T = (b_item + kMarkTile - 1) / kMarkTile; T * kMarkTile < e_item; T++) {
                tile_row[T] = i;
                tile_pos[T] = min(T * kMarkTile - i, re - base);
            }
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
            const int tmax = __reduce_max_sync(kFull, l > 0 ? (unsigned)t0 : 0u);
            if (P == 1) {
                if (__any_sync(kFull, l > 0)) {
                    for (int t = 0; t <= tmax; t++) {
                        const unsigned v = (l > 0 && t <= t0) ? (unsigned)((l + (int64_t(1) << t) - 1) >> t) : 0u;
                        const unsigned long long sv = warp_sum_u31(v);
                        const unsigned hc = __popc(__ballot_sync(kFull, l > 0 && t0 == t));
                        if (lane == t) {
                            accF += sv;
                            accH += hc;
                        }
                    }
                }
            } else {
                const unsigned peers = __match_any_sync(kFull, t0);
                if (t0 < kMaxT && (peers & ((1u << lane) - 1u)) == 0)
                    atomicAdd(&H_s[p * kMaxT + t0], (unsigned long long)__popc(peers));
                if (__any_sync(kFull, l > 0)) {
                    for (int t = 0; t <= tmax; t++) {
                        const unsigned v = (l > 0 && t <= t0) ? (unsigned)((l + (int64_t(1) << t) - 1) >> t) : 0u;
                        const unsigned long long sv = warp_sum_u31(v);
                        if (lane == 0 && sv) atomicAdd(&F_s[p * kMaxT + t], sv);
                    }
                }
            }
            b = e;
        }
    }
    if (P == 1 && lane < kMaxT) {
        if (accH) atomicAdd(&H_s[lane], accH);
        if (accF) atomicAdd(&F_s[lane], accF);
    }
    block_len_stats(mn, mx, sum, sq, st);  // its __syncthreads also orders the H_s / F_s updates
    for (int q = threadIdx.x; q < P * kMaxT; q += blockDim.x) {
        if (H_s[q]) atomicAdd(&st->part[q / kMaxT].H[q % kMaxT], H_s[q]);
        if (F_s[q]) atomicAdd(&st->part[q / kMaxT].F[q % kMaxT], F_s[q]);
    }
}

// Pass 2 -- column marking over merge-path tiles: tile T holds kMarkTile
// items of the sequence (row ends, nonzeros), so at most kMarkTile rows and
// kMarkTile nonzeros, whatever the row lengths (pass 1 wrote each tile's
// first row and position).  The block ORs bit t0 of each nonzero's segment
// into the mask word of its column.  Row of every nonzero: the block counts
// the rows starting at each tile position (empty rows included) and an
// inclusive block scan of those counts maps position -> row (one LDS per
// nonzero).  Nonzeros are read coalesced, kMarkTile / kThreads per thread in
// one batch so the dependent loads overlap, and every (column, bits) pair
// goes out as a fire-and-forget RED after a warp-level merge of equal columns.
// The mask word of column c lives at slot hslot(c) = (c * odd) mod 2^m, a
// bijection on [0, 2^m), 2^m >= K: columns that are hot together on power-law
// inputs (small indices, few set bits) land on different L2 lines and slices.
#ifndef LF_MARK_HASH
#define LF_MARK_HASH 1
#endif
#ifndef LF_MARK_MODE
#define LF_MARK_MODE 3  // tiles of one natural bucket: 3 = block smem filter, then one RED per column;
                        // other tiles: 0 = L2 check then RED, 2 = L1-cached check, 1 / 3 = RED only
#endif
#ifndef LF_MARK_FILTER
#define LF_MARK_FILTER 2048
#endif
#ifndef LF_MARK_FBITS16
#define LF_MARK_FBITS16 0  // 1: filter bits packed two 16-bit halves per word (twice the slots in 48 KB)
#endif
#ifndef LF_MARK_FILTER_ALL
#define LF_MARK_FILTER_ALL 0  // 1: R-MAT-type tiles (several natural buckets) also go through the filter
#endif
constexpr int kMarkFilter = LF_MARK_FILTER;  // direct-mapped (column, bits) slots per block (mode 3)
constexpr uint32_t kFilterEmpty = 0xFFFFFFFFu;
constexpr uint32_t kHashOdd = LF_MARK_HASH ? 0x9E3779B1u : 1u;
__device__ __forceinline__ uint32_t hslot(int32_t c, uint32_t kmask) { return ((uint32_t)c * kHashOdd) & kmask; }
__device__ __forceinline__ uint32_t ld_ca(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.global.ca.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

__global__ void __launch_bounds__(kThreads, LF_MARK_MIN_BLOCKS) stats_mark_kernel(const int64_t *__restrict__ row_ptr,
                                                              const int32_t *__restrict__ col, int64_t n_rows,
                                                              int64_t S, int P,
                                                              const uint8_t *__restrict__ t0seg,
                                                              const int64_t *__restrict__ tile_row,
                                                              const int64_t *__restrict__ tile_pos, int64_t n_tiles,
                                                              uint32_t *__restrict__ mask, uint32_t kmask) {
    __shared__ int32_t cnt[kMarkTile];     // rows starting at a tile position -> inclusive scan
    __shared__ uint8_t rt0[kMarkTile + 1]; // t0 of the tile's rows (P == 1)
    __shared__ int32_t wsum[kThreads / 32];
    constexpr int kFB = LF_MARK_FBITS16 ? kMarkFilter / 2 : kMarkFilter;
    __shared__ uint32_t fkey[kMarkFilter], fbits[kFB];  // block filter of uniform tiles (cleared below)
    constexpr int K = kMarkTile / kThreads;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    __shared__ unsigned s_tmin, s_tmax;  // natural buckets of the tile's non-empty rows (P == 1)
    for (int q = threadIdx.x; q < kMarkTile; q += blockDim.x) cnt[q] = 0;
    if (threadIdx.x == 0) {
        s_tmin = 0xFFFFFFFFu;
        s_tmax = 0u;
    }
    const int64_t base = row_ptr[0];
    const int64_t T = blockIdx.x;
    const int64_t rlo = tile_row[T];
    const int64_t qa = base + tile_pos[T];
    const int64_t rhi = T + 1 < n_tiles ? tile_row[T + 1] : n_rows - 1;
    const int64_t qb = T + 1 < n_tiles ? base + tile_pos[T + 1] : row_ptr[n_rows];
    __syncthreads();
    {
        unsigned lmin = 0xFFFFFFFFu, lmax = 0u;
        constexpr int RU = 8;  // independent row_ptr loads in flight per thread
        for (int64_t r0 = rlo + threadIdx.x; r0 <= rhi; r0 += (int64_t)blockDim.x * RU) {
            int64_t sr[RU], er[RU];
#pragma unroll
            for (int u = 0; u < RU; u++) {
                const int64_t r = r0 + (int64_t)u * blockDim.x;
                sr[u] = r <= rhi ? __ldg(row_ptr + r) - qa : 0;
                er[u] = r <= rhi ? __ldg(row_ptr + r + 1) - qa : 0;
            }
#pragma unroll
            for (int u = 0; u < RU; u++) {
                const int64_t r = r0 + (int64_t)u * blockDim.x;
                if (r > rhi) break;
                if (P == 1) {
                    const unsigned t0 = (unsigned)ceil_log2_i64(max(er[u] - sr[u], (int64_t)1));
                    rt0[r - rlo] = (uint8_t)t0;
                    if (er[u] > sr[u]) {
                        lmin = min(lmin, t0);
                        lmax = max(lmax, t0);
                    }
                }
                if (r > rlo && sr[u] < qb - qa) atomicAdd(&cnt[sr[u]], 1);
            }
        }
        lmin = __reduce_min_sync(kFull, lmin);
        lmax = __reduce_max_sync(kFull, lmax);
        if (lane == 0 && P == 1) {
            atomicMin(&s_tmin, lmin);
            atomicMax(&s_tmax, lmax);
        }
    }
    __syncthreads();
    // every non-empty row of the tile in one natural bucket (banded, stencil,
    // regular rows): every nonzero gets that bit, no position -> row scan
    const bool uni = P == 1 && s_tmin == s_tmax;
    if (LF_MARK_MODE == 3 && (uni || LF_MARK_FILTER_ALL)) {  // only filtered tiles clear the filter
        // (ordered before its use by the __syncthreads after the scan)
        for (int q = threadIdx.x; q < kMarkFilter; q += blockDim.x) {
            fkey[q] = kFilterEmpty;
            if (q < kFB) fbits[q] = 0u;
        }
    }
    if (!uni) {  // inclusive scan of cnt, conflict-free: warp w scans its 512 entries in
       // 32-wide chunks (shuffles), then adds the totals of the warps before it
        constexpr int PER_WARP = kMarkTile / (kThreads / 32);
        int32_t carry = 0;
        for (int j = 0; j < PER_WARP; j += 32) {
            const int idx = warp * PER_WARP + j + lane;
            int32_t x = cnt[idx];
            for (int o = 1; o < 32; o <<= 1) {
                const int32_t y = __shfl_up_sync(kFull, x, o);
                if (lane >= o) x += y;
            }
            cnt[idx] = x + carry;
            carry += __shfl_sync(kFull, x, 31);
        }
        if (lane == 0) wsum[warp] = carry;
        __syncthreads();
        int32_t off = 0;
        for (int w = 0; w < warp; w++) off += wsum[w];
        if (off)
            for (int j = lane; j < PER_WARP; j += 32) cnt[warp * PER_WARP + j] += off;
    }
    __syncthreads();
    int32_t c[K];
    uint32_t bit[K];
#pragma unroll
    for (int k = 0; k < K; k++) {
        const int64_t q = qa + k * kThreads + threadIdx.x;
        c[k] = q < qb ? __ldg(col + q) : -1;
    }
#pragma unroll
    for (int k = 0; k < K; k++) {
        bit[k] = 0;
        if (c[k] < 0) continue;
        if (uni) {
            bit[k] = 1u << s_tmin;
            continue;
        }
        const int rr = cnt[k * kThreads + threadIdx.x];
        if (P == 1) bit[k] = 1u << rt0[rr];
        else bit[k] = 1u << __ldg(t0seg + (rlo + rr) * P + (int)(c[k] / S));
    }
    uint32_t h[K];
#pragma unroll
    for (int k = 0; k < K; k++) h[k] = c[k] >= 0 ? hslot(c[k], kmask) : 0u;
    if (LF_MARK_MODE == 3 && (uni || LF_MARK_FILTER_ALL)) {
        // block-level merge (tiles of one natural bucket: banded / stencil
        // rows, where a tile of ~4096 nonzeros covers ~200 distinct columns):
        // (column, bits) pairs collect in a direct-mapped shared-memory filter
        // (slot = low bits of the column's hashed slot; read first, most are
        // hits); a column colliding with another goes to L2 at once; after
        // the tile every filled slot issues ONE RED.
#pragma unroll
        for (int k = 0; k < K; k++) {
            if (c[k] < 0) continue;
            const int f = (int)(h[k] & (kMarkFilter - 1));
            uint32_t cur = reinterpret_cast<volatile uint32_t *>(fkey)[f];
            if (cur == kFilterEmpty) {
                cur = atomicCAS(&fkey[f], kFilterEmpty, (uint32_t)c[k]);
                if (cur == kFilterEmpty) cur = (uint32_t)c[k];
            }
            if (cur == (uint32_t)c[k] && (!LF_MARK_FBITS16 || bit[k] < 0x10000u)) {
                const int fw = LF_MARK_FBITS16 ? f >> 1 : f;
                const uint32_t fb = LF_MARK_FBITS16 ? bit[k] << ((f & 1) * 16) : bit[k];
                if ((reinterpret_cast<volatile uint32_t *>(fbits)[fw] & fb) != fb) atomicOr(&fbits[fw], fb);
            } else {
                atomicOr(mask + h[k], bit[k]);  // slot taken by another column
            }
        }
        __syncthreads();
        for (int f = threadIdx.x; f < kMarkFilter; f += blockDim.x) {
            const uint32_t key = fkey[f];
            const uint32_t fb = LF_MARK_FBITS16 ? (fbits[f >> 1] >> ((f & 1) * 16)) & 0xFFFFu : fbits[f];
            if (key != kFilterEmpty && fb) atomicOr(mask + hslot((int32_t)key, kmask), fb);
        }
        return;
    }
    // other tiles: one RED per (column, bit) (LF_MARK_MODE 1 everywhere).
    // Reading the mask word first and skipping bits already set (mode 0)
    // issues as many L2 requests and adds a dependent load: slower on B200.
    {
        uint32_t have[K];
#pragma unroll
        for (int k = 0; k < K; k++)
            have[k] = LF_MARK_MODE == 0 ? __ldcg(mask + h[k]) : LF_MARK_MODE == 2 ? ld_ca(mask + h[k]) : 0u;
#pragma unroll
        for (int k = 0; k < K; k++)
#ifdef LF_DIAG_NORED  // diagnostic builds only: the marking pass without its REDs
            if (c[k] >= 0 && (have[k] & bit[k]) != bit[k] && bit[k] == 0x80000000u) atomicOr(mask + h[k], bit[k]);
#else
            if (c[k] >= 0 && (have[k] & bit[k]) != bit[k]) atomicOr(mask + h[k], bit[k]);
#endif
    }
}

// Pass 3 -- one thread per mask SLOT (coalesced loads; the column is the
// inverse of the slot hash, c = s * odd^-1 mod 2^m): Unat[p][t] = #{c : bit t},
// Utop[p][t] = #{c : highest bit >= t}, the latter as a suffix sum of the
// histogram of highest bits.  Warp-aggregated into shared-memory histograms.
__host__ __device__ constexpr uint32_t inv_odd(uint32_t a) {
    uint32_t x = a;  // Newton: x <- x (2 - a x), 5 steps give 32 bits
    for (int i = 0; i < 5; i++) x *= 2u - a * x;
    return x;
}
static_assert(kHashOdd * inv_odd(kHashOdd) == 1u, "hash inverse");

// 32 x 32 bit-matrix transpose across a warp: on return, bit j of lane t's
// word is bit t of lane j's input word (five shuffle-and-swap rounds).
__device__ __forceinline__ uint32_t transpose32(uint32_t x, int lane) {
    const uint32_t lo[5] = {0x0000FFFFu, 0x00FF00FFu, 0x0F0F0F0Fu, 0x33333333u, 0x55555555u};
#pragma unroll
    for (int i = 0, k = 16; i < 5; i++, k >>= 1) {
        const uint32_t y = __shfl_xor_sync(kFull, x, k);
        x = (lane & k) ? (x & ~lo[i]) | ((y & ~lo[i]) >> k) : (x & lo[i]) | ((y & lo[i]) << k);
    }
    return x;
}

__global__ void __launch_bounds__(kThreads) stats_cols_kernel(const uint32_t *__restrict__ mask, int64_t n_cols,
                                                              int64_t S, int P, StatsDev *st, uint32_t kmask) {
    extern __shared__ unsigned long long sh[];  // Un_s[P][32], Hb_s[P][32]
    unsigned long long *Un_s = sh, *Hb_s = sh + P * kMaxT;
    for (int q = threadIdx.x; q < 2 * P * kMaxT; q += blockDim.x) sh[q] = 0;
    __syncthreads();
    const int lane = threadIdx.x & 31;
    int cur_p = -1;
    unsigned long long my_un = 0, my_hb = 0;
    auto flush = [&]() {
        if (cur_p >= 0 && lane < kMaxT) {
            if (my_un) atomicAdd(&Un_s[cur_p * kMaxT + lane], my_un);
            if (my_hb) atomicAdd(&Hb_s[cur_p * kMaxT + lane], my_hb);
        }
        my_un = my_hb = 0;
    };
    const int64_t n_slots = (int64_t)kmask + 1;
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n_slots; base += stride) {
        const int64_t q = base + threadIdx.x;
        uint32_t m = q < n_slots ? __ldcs(mask + q) : 0u;
        const int64_t c = (int64_t)(((uint32_t)q * inv_odd(kHashOdd)) & kmask);
        if (c >= n_cols) m = 0u;  // (a slot of no column holds 0 anyway)
        const int p = m ? (int)(c / S) : -1;
        const int hb = m ? 31 - __clz(m) : -1;
        // columns of one warp may lie in several partitions: group by p.
        // Lane t counts bit t (Unat) and highest bit t (Hb) of the group's
        // columns in registers; they go to shared memory when the partition
        // changes (P = 1: once, after the loop)
        unsigned todo = __ballot_sync(kFull, m != 0);
        while (todo) {
            const int pp = __shfl_sync(kFull, p, __ffs(todo) - 1);
            const bool mine = m != 0 && p == pp;
            todo &= ~__ballot_sync(kFull, mine);
            if (pp != cur_p) {
                flush();
                cur_p = pp;
            }
            // bit-matrix transpose: lane t then holds bit t of every lane's
            // word, so one popc per lane counts the group's columns
            my_un += __popc(transpose32(mine ? m : 0u, lane));
            my_hb += __popc(transpose32(mine ? 1u << hb : 0u, lane));
        }
    }
    flush();
    __syncthreads();
    for (int q = threadIdx.x; q < P * kMaxT; q += blockDim.x) {
        const int p = q / kMaxT, t = q % kMaxT;
        unsigned long long top = 0;  // Utop[t] = sum_{h >= t} Hb[h]
        for (int h = t; h < kMaxT; h++) top += Hb_s[p * kMaxT + h];
        if (Un_s[q]) atomicAdd(&st->part[p].Unat[t], Un_s[q]);
        if (top) atomicAdd(&st->part[p].Utop[t], top);
    }
}

int num_sms() { return sm_count(); }

}  // namespace

size_t stats_scratch_bytes(int64_t n_rows, int64_t nnz, int P) {
    return (((size_t)n_rows * P + 15) & ~size_t(15)) + (size_t)((nnz + n_rows + kMarkTile - 1) / kMarkTile + 1) * 16;
}

uint32_t mask_slots(int64_t n_cols) {
    uint64_t m = 1;
    while ((int64_t)m < n_cols) m <<= 1;
    return (uint32_t)m;
}


namespace {

// Table 2 row-length statistics alone: the features the
// predictor needs BEFORE P is known (section 5.1-5.2), from row_ptr only
// (8 B per row).  One thread per row, warp then block reduction, one set of
// 64-bit atomics per block.  (Used when the statistics pass is too long to
// run speculatively for P = 1, see lf_cell_configure.)
__global__ void __launch_bounds__(kThreads) features_kernel(const int64_t *__restrict__ row_ptr,
                                                            const int32_t *__restrict__ col, int64_t n_rows,
                                                            StatsDev *st, int rows_grid) {
    if ((int)blockIdx.x >= rows_grid) {  // extra blocks: the group / window samples (as stats_rows_kernel)
        __shared__ int32_t hs[8][256];
        const int w = threadIdx.x >> 5;
        group_sample_warp(row_ptr, col, n_rows, st, (int64_t)(blockIdx.x - rows_grid) * 8 + w, hs[w]);
        return;
    }
    unsigned long long mn = ~0ull, mx = 0, sum = 0, sq = 0;
    const int64_t stride = (int64_t)rows_grid * blockDim.x;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n_rows; i += stride) {
        const unsigned long long len = (unsigned long long)(__ldg(row_ptr + i + 1) - __ldg(row_ptr + i));
        mn = min(mn, len);
        mx = max(mx, len);
        sum += len;
        sq += len * len;
    }
    block_len_stats(mn, mx, sum, sq, st);
}

}  // namespace

cudaError_t launch_features(const lf_csr &A, StatsDev *d_stats, cudaStream_t s) {
    if (A.n_rows <= 0) return cudaSuccess;
    const int64_t want = (A.n_rows + kThreads - 1) / kThreads;
    const int grid = (int)std::min<int64_t>(want, (int64_t)num_sms() * 8);
    const bool smp = A.n_rows >= kGroupRows && A.nnz > 0;
    features_kernel<<<grid + (smp ? kGroupSamples / 8 : 0), kThreads, 0, s>>>(A.row_ptr, A.col_ind, A.n_rows,
                                                                             d_stats, grid);
    return cudaGetLastError();
}

cudaError_t launch_stats(const lf_csr &A, int P, StatsDev *d_stats, uint32_t *d_colmask, uint8_t *d_t0seg,
                         cudaStream_t s, bool sample) {
    const int64_t S = A.n_cols > 0 ? (A.n_cols + P - 1) / P : 1;
    const size_t hist = 2 * (size_t)P * kMaxT * sizeof(unsigned long long);
    if (A.n_rows > 0) {
        const int64_t want = (A.n_rows + kThreads - 1) / kThreads;
#ifndef LF_STATS_ROWS_BPS
#define LF_STATS_ROWS_BPS 8  // stats_rows_kernel grid: at most this many blocks per SM (grid-stride over rows)
#endif
        const int grid = (int)std::min<int64_t>(want, (int64_t)num_sms() * LF_STATS_ROWS_BPS);
        const int64_t tiles = (A.nnz + A.n_rows + kMarkTile - 1) / kMarkTile;
        if (tiles > 0x7fffffff) return cudaErrorInvalidValue;
        int64_t *tile_row = reinterpret_cast<int64_t *>(d_t0seg + (((size_t)A.n_rows * P + 15) & ~size_t(15)));
        int64_t *tile_pos = tile_row + tiles;
        const bool smp = sample && A.n_rows >= kGroupRows && A.nnz > 0;
        stats_rows_kernel<<<grid + (smp ? kGroupSamples / 8 : 0), kThreads, hist, s>>>(
            A.row_ptr, A.col_ind, A.n_rows, S, P, d_stats, d_t0seg, tile_row, tile_pos, grid);
        if (A.nnz > 0)
            stats_mark_kernel<<<(unsigned)tiles, kThreads, 0, s>>>(A.row_ptr, A.col_ind, A.n_rows, S, P, d_t0seg,
                                                                    tile_row, tile_pos, tiles, d_colmask,
                                                                    mask_slots(A.n_cols) - 1);
    }
    if (A.n_cols > 0) {
        const int64_t want = ((int64_t)mask_slots(A.n_cols) + kThreads - 1) / kThreads;
        const int grid = (int)std::min<int64_t>(want, (int64_t)num_sms() * 8);
        stats_cols_kernel<<<grid, kThreads, hist, s>>>(d_colmask, A.n_cols, S, P, d_stats, mask_slots(A.n_cols) - 1);
    }
    return cudaGetLastError();
}

}  // namespace lf
