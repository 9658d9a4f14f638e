// cell_spmm.cu -- CELL SpMM C = A . B on sm_100a.
//
// PAPER.md Alg. 2 per CELL row:  i = rowInd[r];
//   local[j] = sum_w val[r][w] * B[colInd[r][w]][j];  C[i][j] (+)= local[j].
// B200 mapping:
//   * a WARP TASK is 32 consecutive slots of a bucket with W <= 32 (32/W whole
//     CELL rows: one 2^k-slot block when k = 5), or one CELL row when W > 32;
//     warps take CH consecutive tasks per round (chunked grid-stride), so the
//     whole grid sweeps the buckets partition-major and each warp streams
//     colInd/val with coalesced 128-byte loads, prefetching the next task's
//     slots and row tags while it gathers the current one;
//   * the lanes split J: J/4 float4 columns over 32/G lanes, G lane groups
//     each taking every G-th slot (G = 4, 2, 1 for J <= 32, 64, >= 128); NV
//     float4 per lane cover J up to 512 per pass (J tiles beyond that);
//   * each 32-slot chunk is staged by cp.async and resolved once into B-row
//     addresses + values in shared memory (broadcast reads); B rows are
//     gathered as float4 through the read-only path, U slots in flight per lane;
//   * the index/value/tag streams and C stores carry an L2 evict_first policy
//     so the L2 keeps B rows;
//   * the row width W is a template parameter for W <= 32, so the fold /
//     group reduction and the C update positions are compile-time;
//   * folded rows (reading R4: consecutive CELL rows of one source row) are
//     summed in registers across consecutive tasks of a warp; a run that holds
//     every CELL row of its source row is written with a plain vector store,
//     otherwise (run split between warps, or P > 1) red.global.add.v4.f32 into
//     the row zeroed beforehand by zero_rows_kernel (reading R11);
//   * rows of A with no CELL row are zeroed by zero_rows_kernel (R13).
// Alternative executions of the same CELL arrays (chosen per handle, below):
// the grouped path (4 CELL rows per warp, one gather per distinct column) and
// its tensor-core variant (opt-in); C is the same up to fp32 summation order.
// Row tag (built by bucket_kernel<1>): (i << 3) | S<<2 | F<<1 | L, where F/L
// mark the first/last sub-row of the (row, partition) segment and S that the
// segment holds all of the row's CELL rows; -1 = padding row.
#include "cell_spmm_impl.cuh"

namespace lf {

// rows written with red.global.add must be zero first: kRowRed always, and
// kRowRun rows too when J needs several tiles (no run merging then)
cudaError_t zero_red_rows(const SpmmArgs &a, bool tiled, cudaStream_t s) {
    if (a.n_rows == 0 || a.J == 0) return cudaSuccess;
    const int vec4 = (a.J % 4 == 0 && a.ldc % 4 == 0 && (a.c_bits & 15) == 0) ? 1 : 0;
    const unsigned mask = (1u << kRowRed) | (tiled ? (1u << kRowRun) : 0u) | (LF_EPI_ZERO ? 0u : (1u << kRowEmpty));
    int64_t warps = (a.n_rows + 31) / 32;
    int grid = (int)std::max<int64_t>(1, std::min<int64_t>((warps + 7) / 8, (int64_t)sm_count() * 16));
    zero_rows_kernel<<<grid, 256, 0, s>>>(a.row_mode, a.n_rows, a.C, a.ldc, a.J, vec4, mask, a.n_dst, a.dst,
                                          a.row_base);
    return cudaGetLastError();
}

bool grouped_ok(const SpmmArgs &a) {
    return a.grouped && a.nb_g > 0 && vec4_ok(a.B, a.ldb, a.c_bits, a.ldc, a.J) && a.J <= 128;
}

bool mma_ok(const SpmmArgs &a) {
    return a.mma && a.n_dst == 0 && a.nb_g > 0 && vec4_ok(a.B, a.ldb, a.c_bits, a.ldc, a.J) && a.J % 64 == 0 &&
           a.J <= 128;
}

const char *cell_spmm_path(const SpmmArgs &a) {
    if (a.J == 0 || a.n_rows == 0) return "";
    if (tc_ok(a)) return "cell_spmm_tc_kernel";
    if (mma_ok(a)) return "cell_spmm_mma_kernel";
    if (grouped_ok(a)) return "cell_spmm_grouped_kernel";
    return "cell_spmm_kernel";
}

cudaError_t launch_cell_spmm(const SpmmArgs &a, cudaStream_t s) {
    if (a.J == 0 || a.n_rows == 0) return cudaSuccess;
    const bool v4 = vec4_ok(a.B, a.ldb, a.c_bits, a.ldc, a.J);
    if (tc_ok(a)) {  // runs of folded rows are split across groups: red.add, pre-zeroed
        cudaError_t e = zero_red_rows(a, true, s);
        if (e != cudaSuccess) return e;
        return launch_cell_spmm_tc(a, s);
    }
    if (mma_ok(a)) {
        cudaError_t e = zero_red_rows(a, true, s);
        if (e != cudaSuccess) return e;
        return spmm_mma(a, s);
    }
    if (a.n_dst > 0) {  // fused row exchange: the destination-writing instantiations (cell_spmm_md.cu)
        const bool tiled = a.J > 128;  // spmm_md's kernels pass 128 columns at a time
        cudaError_t e = zero_red_rows(a, grouped_ok(a) || tiled, s);
        if (e != cudaSuccess) return e;
        return spmm_md(a, v4, s);
    }
    if (grouped_ok(a)) {  // runs of folded rows are split across groups: red.add, pre-zeroed
        cudaError_t e = zero_red_rows(a, true, s);
        if (e != cudaSuccess) return e;
        return spmm_grouped(a, s);
    }
    const bool tiled = v4 ? a.J > 512 : a.J > 128;
    cudaError_t e = zero_red_rows(a, tiled, s);
    if (e != cudaSuccess) return e;
#ifndef LF_VEC8
#define LF_VEC8 1  // 256-bit B-row gathers where J % 8 == 0 and B / C rows are 32-byte aligned
#endif
    // measured: c2 J = 128 0.603 -> 0.592 ms, c4 J = 256 6.01 -> 5.76 ms; J = 64 slower (0.363 -> 0.390)
    if (LF_VEC8 && vec8_ok(a.B, a.ldb, a.c_bits, a.ldc, a.J) && a.J > 64) return spmm_v8(a, s);
    if (v4) {
        if (a.J <= 32) return run_cell_j<4, 4, 1>(a, s);
        if (a.J <= 64) return run_cell_j<4, 2, 1>(a, s);
        if (a.J <= 128) return run_cell_j<4, 1, 1>(a, s);
        if (a.J <= 256) return run_cell_j<4, 1, 2>(a, s);
        return run_cell_j<4, 1, 4>(a, s);
    }
    return run_cell<1, 1, 4, false>(a, s);
}

cudaError_t launch_csr_spmm(const lf_csr &A, const float *B, int64_t ldb, int J, float *C, int64_t ldc,
                            cudaStream_t s) {
    if (A.n_rows == 0 || J == 0) return cudaSuccess;
    if (vec4_ok(B, ldb, C, ldc, J)) {
        if (J <= 32) return run_csr_j<4, 4, 1>(A, B, ldb, J, C, ldc, s);
        if (J <= 64) return run_csr_j<4, 2, 1>(A, B, ldb, J, C, ldc, s);
        if (J <= 128) return run_csr_j<4, 1, 1>(A, B, ldb, J, C, ldc, s);
        if (J <= 256) return run_csr_j<4, 1, 2>(A, B, ldb, J, C, ldc, s);
        return run_csr_j<4, 1, 4>(A, B, ldb, J, C, ldc, s);
    }
    return run_csr<1, 1, 4, false>(A, B, ldb, J, C, ldc, s);
}

}  // namespace lf
