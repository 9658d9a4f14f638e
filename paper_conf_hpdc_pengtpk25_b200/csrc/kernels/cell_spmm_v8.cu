// cell_spmm_v8.cu -- the per-slot CELL SpMM kernels with 256-bit B-row
// gathers (ld.global.nc.v8.f32, J > 64, 32-byte aligned B / C rows); kernels in
// cell_spmm_impl.cuh, dispatch in cell_spmm.cu (own translation unit so nvcc
// compiles the instantiations in parallel).
#include "cell_spmm_impl.cuh"

namespace lf {

cudaError_t spmm_v8(const SpmmArgs &a, cudaStream_t s) {
    if (a.J <= 128) return run_cell_j<8, 2, 1>(a, s);
    if (a.J <= 256) return run_cell_j<8, 1, 1>(a, s);
    return run_cell_j<8, 1, 2>(a, s);
}

}  // namespace lf
