/*
 * lf_oracle.c -- TEST INFRASTRUCTURE ONLY.  The plain, slow, obviously-correct
 * CPU statement of what LiteForm's hot path computes.  Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference leg
 * may load it.  It shares no code, header or constant with the CUDA path
 * (paper_conf_hpdc_pengtpk25_b200/csrc) and neither side includes the other.
 *
 * Citations: P:L<a>-<b> = /root/reference/PAPER.md lines a-b (PDF-extracted
 * text of Peng et al., "LiteForm", HPDC'25).  Readings of garbled / silent
 * passages are SURVEY.md 8(c) C1-C17, restated in DESIGN.md "Readings".
 *
 * Pinned by tests/test_oracle_*.py:
 *   lfo_spmm_csr          dense GEMM on tiny integer inputs, A=I, diagonal/permutation
 *   lfo_csr_to_cell       lossless CELL->CSR round trip, invariants, closed forms
 *                         (regular rows, 27-point stencil census)
 *   lfo_cell_to_csr       round trip
 *   lfo_cell_spmm         == lfo_spmm_csr exactly on integer inputs
 *   lfo_partition_cost    hand-worked eq.7 examples (tests/golden/cost_*.txt)
 *   lfo_partition_stats   definitions restated through lfo_partition_cost
 *   lfo_build_buckets     brute-force argmin when the cost is unimodal,
 *                         separating example (golden)
 *   lfo_features          numpy statistics of the row lengths
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* ---------------------------------------------------------------------- */
/* Algorithm 1, eq. 3:                            */
/*   C[i][j] = sum_{pos=rowPtr[i]}^{rowPtr[i+1]-1} val[pos] * B[colInd[pos]][j] */
/* accumulated in fp64.  The (i, j, pos) loops are run as (i, pos, j) with   */
/* one fp64 accumulator per (i,j); every C[i][j] still sums pos in ascending */
/* order, i.e. the same additions in the same order as Alg. 1.              */
/* Cabs[i][j] = sum |val[pos]| * |B[k][j]|, the scale of the tolerance       */
/* (BASELINE.json north_star: |C - C_ref| <= 1e-5 * (|A|.|B|)).             */
/* rows[] (optional, n_out entries) selects which rows to compute; NULL = all */
/* ---------------------------------------------------------------------- */
void lfo_spmm_csr(int64_t n_out, const int64_t *rows, int64_t J, const int64_t *rowPtr, const int32_t *colInd,
                  const float *val, const float *B, int64_t ldb, double *C, double *Cabs) {
#pragma omp parallel for schedule(dynamic, 16)
    for (int64_t o = 0; o < n_out; o++) {
        int64_t i = rows ? rows[o] : o;
        double *c = C + o * J;
        double *ca = Cabs ? Cabs + o * J : NULL;
        for (int64_t j = 0; j < J; j++) {
            c[j] = 0.0;
            if (ca) ca[j] = 0.0;
        }
        for (int64_t pos = rowPtr[i]; pos < rowPtr[i + 1]; pos++) {
            int64_t k = colInd[pos];
            double a = (double)val[pos];
            const float *b = B + k * ldb;
            for (int64_t j = 0; j < J; j++) {
                c[j] += a * (double)b[j];
                if (ca) ca[j] += fabs(a) * fabs((double)b[j]);
            }
        }
    }
}

/* smallest t with 2^t >= l  (l >= 1): the natural bucket, 2^(t-1) < l <= 2^t
 * (reading C1 of P:L494-497, L814-817, L993-995; Fig. 3 labels L507-520) */
static int ceil_log2(int64_t l) {
    int t = 0;
    while (((int64_t)1 << t) < l) t++;
    return t;
}

/* Column partition p of P over K columns: "evenly divides the columns"
 * (P:L490-491), reading C3: S = ceil(K/P), partition p = [p*S, min(p*S+S, K)).
 * Segment of row i in partition p: positions [*beg, *end) of the row whose
 * column lies in the partition (columns are sorted within the row). */
static void segment(const int64_t *rowPtr, const int32_t *colInd, int64_t i, int64_t K, int32_t P, int32_t p,
                    int64_t *beg, int64_t *end) {
    int64_t S = (K + P - 1) / P;
    int64_t lo = (int64_t)p * S, hi = lo + S < K ? lo + S : K;
    int64_t b = rowPtr[i];
    while (b < rowPtr[i + 1] && colInd[b] < lo) b++;
    int64_t e = b;
    while (e < rowPtr[i + 1] && colInd[e] < hi) e++;
    *beg = b;
    *end = e;
}

typedef struct {
    int32_t part;           /* partition p */
    int32_t width_log2;     /* t: bucket width W = 2^t */
    int32_t rows_per_block; /* R_t = 2^(k_p - t) */
    int32_t pad_;
    int64_t n_rows;     /* CELL rows holding data (folded rows counted per sub-row) */
    int64_t n_rows_pad; /* n_rows rounded up to a multiple of R_t */
    int64_t row_off;    /* first CELL row of the bucket in rowInd */
    int64_t slot_off;   /* first slot of the bucket in colInd/val */
} lfo_bucket;

/* ---------------------------------------------------------------------- */
/* CSR -> CELL (section 4, Fig. 3/4, folding P:L832-843).        */
/* Step by step, readings C1-C7:                                            */
/*  for p ascending; for bucket t = 0..e_p ascending (width 2^t);            */
/*   for row i ascending: l = |segment of row i in p|; skip l = 0;           */
/*     t_i = min(ceil_log2(l), e_p)  -- rows longer than W_p=2^e_p go to the */
/*       max bucket as folded rows (C4);                                    */
/*     if t_i == t: append n_sub = ceil(l / 2^t) CELL rows, each with       */
/*       rowInd = i, holding the next 2^t entries of the segment in CSR      */
/*       order; missing slots = (colInd -1, val +0.0f)  (C5, C6)             */
/*   pad the bucket to a multiple of R_t = 2^(k_p - t) rows with rowInd=-1  */
/*   (blocks of 2^k_p slots; C2); omit empty buckets. */
/* Buckets are concatenated partition-major, ascending width (C7).          */
/* If out arrays are NULL only the sizes are returned.                      */
/* Returns 0, or -1 on a bad parameter.                                     */
/* ---------------------------------------------------------------------- */
int lfo_csr_to_cell(int64_t I, int64_t K, const int64_t *rowPtr, const int32_t *colInd, const float *val,
                    int32_t P, const int8_t *e, const int8_t *k, int64_t *R_tot, int64_t *S_tot,
                    int32_t *n_buckets, int32_t *rowInd, int32_t *colIndC, float *valC, lfo_bucket *buckets) {
    if (P < 1) return -1;
    for (int32_t p = 0; p < P; p++)
        if (e[p] < 0 || e[p] > 30 || k[p] < e[p] || k[p] > 30) return -1;
    int64_t r = 0, s = 0;
    int32_t nb = 0;
    for (int32_t p = 0; p < P; p++) {
        for (int t = 0; t <= e[p]; t++) {
            int64_t W = (int64_t)1 << t;
            int64_t R = (int64_t)1 << (k[p] - t);
            int64_t count = 0, r0 = r, s0 = s;
            for (int64_t i = 0; i < I; i++) {
                int64_t beg, end;
                segment(rowPtr, colInd, i, K, P, p, &beg, &end);
                int64_t l = end - beg;
                if (l == 0) continue;
                int ti = ceil_log2(l);
                if (ti > e[p]) ti = e[p];
                if (ti != t) continue;
                int64_t n_sub = (l + W - 1) / W;
                for (int64_t sub = 0; sub < n_sub; sub++) {
                    if (rowInd) rowInd[r] = (int32_t)i;
                    for (int64_t w = 0; w < W; w++) {
                        int64_t q = sub * W + w;
                        if (colIndC) {
                            if (q < l) {
                                colIndC[s] = colInd[beg + q];
                                valC[s] = val[beg + q];
                            } else {
                                colIndC[s] = -1;
                                valC[s] = 0.0f;
                            }
                        }
                        s++;
                    }
                    r++;
                    count++;
                }
            }
            if (count == 0) continue;
            int64_t padded = (count + R - 1) / R * R;
            for (int64_t q = count; q < padded; q++) {
                if (rowInd) rowInd[r] = -1;
                for (int64_t w = 0; w < W; w++) {
                    if (colIndC) {
                        colIndC[s] = -1;
                        valC[s] = 0.0f;
                    }
                    s++;
                }
                r++;
            }
            if (buckets) {
                lfo_bucket *b = &buckets[nb];
                b->part = p;
                b->width_log2 = t;
                b->rows_per_block = (int32_t)R;
                b->pad_ = 0;
                b->n_rows = count;
                b->n_rows_pad = padded;
                b->row_off = r0;
                b->slot_off = s0;
            }
            nb++;
        }
    }
    *R_tot = r;
    *S_tot = s;
    *n_buckets = nb;
    return 0;
}

/* ---------------------------------------------------------------------- */
/* CELL -> CSR, the inverse: collect every real slot (colInd >= 0) as       */
/* (row, col, val) in CELL order, then stable-sort by (row, col) (insertion */
/* sort per row).  rowPtr_out[I+1], colInd_out/val_out sized S_tot.          */
/* Returns nnz, or -1 if a real slot sits in a padding row.                 */
/* ---------------------------------------------------------------------- */
int64_t lfo_cell_to_csr(int64_t I, int32_t n_buckets, const lfo_bucket *buckets, const int32_t *rowInd,
                        const int32_t *colIndC, const float *valC, int64_t *rowPtr_out, int32_t *colInd_out,
                        float *val_out) {
    for (int64_t i = 0; i <= I; i++) rowPtr_out[i] = 0;
    /* count */
    for (int32_t b = 0; b < n_buckets; b++) {
        int64_t W = (int64_t)1 << buckets[b].width_log2;
        for (int64_t q = 0; q < buckets[b].n_rows_pad; q++) {
            int64_t r = buckets[b].row_off + q;
            for (int64_t w = 0; w < W; w++) {
                int64_t s = buckets[b].slot_off + q * W + w;
                if (colIndC[s] < 0) continue;
                if (rowInd[r] < 0 || rowInd[r] >= I) return -1;
                rowPtr_out[rowInd[r] + 1]++;
            }
        }
    }
    for (int64_t i = 0; i < I; i++) rowPtr_out[i + 1] += rowPtr_out[i];
    int64_t *fill = (int64_t *)malloc((size_t)(I + 1) * sizeof(int64_t));
    if (!fill) return -1;
    memcpy(fill, rowPtr_out, (size_t)(I + 1) * sizeof(int64_t));
    for (int32_t b = 0; b < n_buckets; b++) {
        int64_t W = (int64_t)1 << buckets[b].width_log2;
        for (int64_t q = 0; q < buckets[b].n_rows_pad; q++) {
            int64_t r = buckets[b].row_off + q;
            for (int64_t w = 0; w < W; w++) {
                int64_t s = buckets[b].slot_off + q * W + w;
                if (colIndC[s] < 0) continue;
                int64_t d = fill[rowInd[r]]++;
                colInd_out[d] = colIndC[s];
                val_out[d] = valC[s];
            }
        }
    }
    free(fill);
    /* stable insertion sort by column inside every row */
    for (int64_t i = 0; i < I; i++) {
        for (int64_t a = rowPtr_out[i] + 1; a < rowPtr_out[i + 1]; a++) {
            int32_t c = colInd_out[a];
            float v = val_out[a];
            int64_t q = a - 1;
            while (q >= rowPtr_out[i] && colInd_out[q] > c) {
                colInd_out[q + 1] = colInd_out[q];
                val_out[q + 1] = val_out[q];
                q--;
            }
            colInd_out[q + 1] = c;
            val_out[q + 1] = v;
        }
    }
    return rowPtr_out[I];
}

/* ---------------------------------------------------------------------- */
/* Algorithm 2, eq. 4, fp64, over every block of  */
/* every bucket:  i = rowInd[iBlk]; local = sum_kBlk val*B[colInd][j];       */
/* C[i][j] += local.  Padding rows (rowInd<0) and padding slots (colInd<0)  */
/* are skipped (reading C12); C starts at 0 (C13: C = A.B).                  */
/* ---------------------------------------------------------------------- */
void lfo_cell_spmm(int64_t I, int64_t J, int32_t n_buckets, const lfo_bucket *buckets, const int32_t *rowInd,
                   const int32_t *colIndC, const float *valC, const float *B, int64_t ldb, double *C) {
    /* Threads split the j range (the output columns): every thread walks all
     * blocks in Alg. 2's order for its own columns, so each C[i][j] receives
     * the same additions in the same order whatever the thread count. */
#pragma omp parallel
    {
        int64_t nt = 1, id = 0;
#ifdef _OPENMP
        nt = omp_get_num_threads();
        id = omp_get_thread_num();
#endif
        const int64_t j0 = J * id / nt, j1 = J * (id + 1) / nt;
        for (int64_t i = 0; i < I; i++)
            for (int64_t j = j0; j < j1; j++) C[i * J + j] = 0.0;
        for (int32_t b = 0; b < n_buckets && j0 < j1; b++) {
            int64_t W = (int64_t)1 << buckets[b].width_log2;
            int64_t R = buckets[b].rows_per_block;
            int64_t n_blocks = buckets[b].n_rows_pad / R;
            for (int64_t blk = 0; blk < n_blocks; blk++) {
                for (int64_t iBlk = 0; iBlk < R; iBlk++) {
                    int64_t r = buckets[b].row_off + blk * R + iBlk;
                    int64_t i = rowInd[r];
                    if (i < 0) continue;
                    for (int64_t j = j0; j < j1; j++) {
                        double local = 0.0;
                        for (int64_t kBlk = 0; kBlk < W; kBlk++) {
                            int64_t s = buckets[b].slot_off + (blk * R + iBlk) * W + kBlk;
                            int64_t kk = colIndC[s];
                            if (kk < 0) continue;
                            local += (double)valC[s] * (double)B[kk * ldb + j];
                        }
                        C[i * J + j] += local;
                    }
                }
            }
        }
    }
}

/* ---------------------------------------------------------------------- */
/* Eq. 7, reading C10, for partition p with max bucket width 2^e:  */
/*   cost = sum over the partition's buckets x of                           */
/*          2 * I1(x) * W(x) + |set(Ind(x))| * J + I1(x) * J                  */
/* I1 = CELL rows of the bucket including folded rows, excluding block       */
/* padding (Alg. 3 runs before blocks exist); set(Ind) = distinct column     */
/* indices held by the bucket.  The buckets are MATERIALISED    */
/* as in lfo_csr_to_cell (TuneWidth) and the distinct columns  */
/* are counted with an explicit set (stamp array).  Exact int64.            */
/* Returns -1 if e is out of range.                                         */
/* ---------------------------------------------------------------------- */
int64_t lfo_partition_cost(int64_t I, int64_t K, const int64_t *rowPtr, const int32_t *colInd, int32_t P,
                           int32_t p, int32_t e, int64_t J) {
    if (e < 0 || e > 30) return -1;
    int64_t total = 0;
    int failed = 0;
    /* the buckets t = 0..e are independent sets: one thread (and one stamp
     * array) per bucket; the int64 sum does not depend on the order */
#pragma omp parallel for schedule(dynamic, 1) reduction(+ : total, failed)
    for (int t = 0; t <= e; t++) {
        char *seen = (char *)calloc((size_t)(K > 0 ? K : 1), 1);
        if (!seen) {
            failed++;
            continue;
        }
        int64_t W = (int64_t)1 << t;
        int64_t I1 = 0, U = 0;
        for (int64_t i = 0; i < I; i++) {
            int64_t beg, end;
            segment(rowPtr, colInd, i, K, P, p, &beg, &end);
            int64_t l = end - beg;
            if (l == 0) continue;
            int ti = ceil_log2(l);
            if (ti > e) ti = e;
            if (ti != t) continue;
            I1 += (l + W - 1) / W;
            for (int64_t q = beg; q < end; q++) {
                if (!seen[colInd[q]]) {
                    seen[colInd[q]] = 1;
                    U++;
                }
            }
        }
        free(seen);
        if (I1 == 0) continue;
        total += 2 * I1 * W + U * J + I1 * J;
    }
    return failed ? -1 : total;
}

/* Largest natural bucket of partition p: ceil_log2(max segment length), or
 * -1 for an all-empty partition (reading C9: rW = max width in buckets,
 * P:L920; an empty partition has no buckets). */
int32_t lfo_partition_max_log2(int64_t I, int64_t K, const int64_t *rowPtr, const int32_t *colInd, int32_t P,
                               int32_t p) {
    int64_t mx = 0;
    for (int64_t i = 0; i < I; i++) {
        int64_t beg, end;
        segment(rowPtr, colInd, i, K, P, p, &beg, &end);
        if (end - beg > mx) mx = end - beg;
    }
    return mx == 0 ? -1 : ceil_log2(mx);
}

/* ---------------------------------------------------------------------- */
/* Algorithm 3, BuildBuckets (prose L991-1006), read in         */
/* EXPONENT space (reading C8): lo = 0 (lW = 2^0 = 1, line 4),               */
/* hi = log2 rW (line 3); while lo < hi: mid = (lo+hi)/2 (line 6);           */
/* if cost(2^mid) > cost(2^(mid+1)) (line 11) lo = mid+1 (line 12: lW=2*mW)  */
/* else hi = mid (line 14); return 2^lo (line 15).                           */
/* Returns e = log2 of the chosen max width, or -1 for an empty partition.  */
/* ---------------------------------------------------------------------- */
int32_t lfo_build_buckets(int64_t I, int64_t K, const int64_t *rowPtr, const int32_t *colInd, int32_t P,
                          int32_t p, int64_t J) {
    int32_t hi = lfo_partition_max_log2(I, K, rowPtr, colInd, P, p);
    if (hi < 0) return -1;
    int32_t lo = 0;
    while (lo < hi) {
        int32_t mid = (lo + hi) / 2;
        int64_t mCost = lfo_partition_cost(I, K, rowPtr, colInd, P, p, mid, J);
        int64_t mCost2 = lfo_partition_cost(I, K, rowPtr, colInd, P, p, mid + 1, J);
        if (mCost > mCost2) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

/* Algorithm 3 read LITERALLY in width space: lW = 1,
 * rW = max width; mW = (lW + rW)/2 with integer division.  Kept only to
 * document reading C8 (tests show where it differs).  Returns the WIDTH. */
int64_t lfo_build_buckets_literal(int64_t I, int64_t K, const int64_t *rowPtr, const int32_t *colInd, int32_t P,
                                  int32_t p, int64_t J) {
    int32_t top = lfo_partition_max_log2(I, K, rowPtr, colInd, P, p);
    if (top < 0) return -1;
    int64_t lW = 1, rW = (int64_t)1 << top;
    while (lW < rW) {
        int64_t mW = (lW + rW) / 2;
        int32_t em = ceil_log2(mW);
        if (((int64_t)1 << em) != mW) return -2; /* never happens: mW stays a power of two */
        int64_t mCost = lfo_partition_cost(I, K, rowPtr, colInd, P, p, em, J);
        int64_t mCost2 = lfo_partition_cost(I, K, rowPtr, colInd, P, p, em + 1, J);
        if (mCost > mCost2) lW = 2 * mW;
        else rW = mW;
    }
    return lW;
}

/* ---------------------------------------------------------------------- */
/* Per-partition bucket statistics, straight from their definitions with    */
/* explicit sets (t = natural bucket t0 = ceil_log2 l of a row segment):    */
/*   H[t]    = #segments with t0 == t                                       */
/*   F[t]    = sum over segments with t0 >= t of ceil(l / 2^t)               */
/*   Unat[t] = |union of the columns of segments with t0 == t|               */
/*   Utop[t] = |union of the columns of segments with t0 >= t|               */
/* With these, eq. 7 for max width 2^e is                                   */
/*   sum_{b<e, H[b]>0} (2 H[b] 2^b + Unat[b] J + H[b] J)                     */
/*   + (F[e] > 0 ? 2 F[e] 2^e + Utop[e] J + F[e] J : 0)                      */
/* (tests check this identity against lfo_partition_cost).  Arrays of 32.   */
/* ---------------------------------------------------------------------- */
void lfo_partition_stats(int64_t I, int64_t K, const int64_t *rowPtr, const int32_t *colInd, int32_t P, int32_t p,
                         int64_t *H, int64_t *F, int64_t *Unat, int64_t *Utop) {
    int32_t *stamp = (int32_t *)calloc((size_t)(K > 0 ? K : 1), sizeof(int32_t));
    for (int t = 0; t < 32; t++) {
        H[t] = F[t] = Unat[t] = Utop[t] = 0;
        int32_t tagN = 2 * t + 1, tagT = 2 * t + 2;
        /* Unat pass */
        for (int64_t i = 0; i < I; i++) {
            int64_t beg, end;
            segment(rowPtr, colInd, i, K, P, p, &beg, &end);
            int64_t l = end - beg;
            if (l == 0) continue;
            int t0 = ceil_log2(l);
            if (t0 == t) {
                H[t]++;
                for (int64_t q = beg; q < end; q++)
                    if (stamp[colInd[q]] != tagN) { stamp[colInd[q]] = tagN; Unat[t]++; }
            }
        }
        /* Utop pass */
        for (int64_t i = 0; i < I; i++) {
            int64_t beg, end;
            segment(rowPtr, colInd, i, K, P, p, &beg, &end);
            int64_t l = end - beg;
            if (l == 0) continue;
            int t0 = ceil_log2(l);
            if (t0 >= t) {
                F[t] += (l + ((int64_t)1 << t) - 1) >> t;
                for (int64_t q = beg; q < end; q++)
                    if (stamp[colInd[q]] != tagT) { stamp[colInd[q]] = tagT; Utop[t]++; }
            }
        }
    }
    free(stamp);
}

/* ---------------------------------------------------------------------- */
/* Table 2 features of the row lengths l_i, fp64, two-pass:     */
/*  out[0..6] = n_rows, n_cols, nnz, mean, min, max, population std.        */
/* Table 3 = the same over densities l_i / K, plus J.           */
/* ---------------------------------------------------------------------- */
void lfo_features(int64_t I, int64_t K, const int64_t *rowPtr, double *out) {
    int64_t nnz = rowPtr[I] - rowPtr[0];
    int64_t mn = I > 0 ? rowPtr[1] - rowPtr[0] : 0, mx = mn;
    for (int64_t i = 0; i < I; i++) {
        int64_t l = rowPtr[i + 1] - rowPtr[i];
        if (l < mn) mn = l;
        if (l > mx) mx = l;
    }
    double mean = I > 0 ? (double)nnz / (double)I : 0.0;
    double ss = 0.0;
    for (int64_t i = 0; i < I; i++) {
        double d = (double)(rowPtr[i + 1] - rowPtr[i]) - mean;
        ss += d * d;
    }
    out[0] = (double)I;
    out[1] = (double)K;
    out[2] = (double)nnz;
    out[3] = mean;
    out[4] = (double)mn;
    out[5] = (double)mx;
    out[6] = I > 0 ? sqrt(ss / (double)I) : 0.0;
}

/* Thread count of the OpenMP loops above (tests check thread-count
 * independence; bench.py's cpu_baseline reports the count it used). */
int32_t lfo_set_threads(int32_t n) {
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
    return omp_get_max_threads();
#else
    (void)n;
    return 1;
#endif
}
