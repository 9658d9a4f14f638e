// cell_spmm_grp.cu -- instantiations of the grouped (column-merged, 4-row
// groups) and mma.sync grouped CELL SpMM kernels; kernels in
// cell_spmm_impl.cuh, dispatch in cell_spmm.cu.
#include "cell_spmm_impl.cuh"

namespace lf {

cudaError_t spmm_grouped(const SpmmArgs &a, cudaStream_t s) {
    if (a.J <= 32) return run_grouped_j<4, 1>(a, s);
    if (a.J <= 64) return run_grouped_j<2, 1>(a, s);
    return run_grouped_j<1, 1>(a, s);
}

cudaError_t spmm_mma(const SpmmArgs &a, cudaStream_t s) { return run_mma<8>(a, s); }

}  // namespace lf
