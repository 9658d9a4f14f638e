// cell_spmm_md.cu -- the fused-row-exchange instantiations (lf_spmm_ex with
// destinations): per-slot and grouped kernels whose C-row writes go to every
// destination C (MD = true; no full-tile variants).  Kernels in
// cell_spmm_impl.cuh, dispatch (and the pre-zeroing) in cell_spmm.cu.
#include "cell_spmm_impl.cuh"

namespace lf {

cudaError_t spmm_md(const SpmmArgs &a, bool v4, cudaStream_t s) {
    // one instantiation per kernel family: 128-column passes (J > 128 in tiles,
    // J < 128 with idle lanes) -- this path trades a little speed for
    // compile time; the caller pre-zeroes run rows when J > 128 (tiled)
    if (grouped_ok(a)) return run_grouped<1, 1, false, true>(a, s);
    if (v4) return run_cell<4, 1, 1, false, true>(a, s);
    return run_cell<1, 1, 4, false, true>(a, s);
}

}  // namespace lf
