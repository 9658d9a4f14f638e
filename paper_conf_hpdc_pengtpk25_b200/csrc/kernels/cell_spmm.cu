// cell_spmm.cu -- CELL SpMM C = A . B on sm_100a.
//
// PAPER.md Alg. 2 per CELL row:  i = rowInd[r];
//   local[j] = sum_w val[r][w] * B[colInd[r][w]][j];  C[i][j] (+)= local[j].
// B200 mapping:
//   * a WARP TASK is 32 consecutive slots of a bucket with W <= 32 (32/W whole
//     CELL rows: one 2^k-slot block when k = 5), or one CELL row when W > 32;
//     tasks are contiguous in slot order, so warps stream colInd/val with one
//     coalesced 128-byte load each and walk buckets partition-major;
//   * the lanes split J: J/4 float4 columns over 32/G lanes, G lane groups
//     each taking every G-th slot (G = 4, 2, 1 for J <= 32, 64, >= 128); NV
//     float4 per lane cover J up to 512 per pass (J tiles beyond that);
//   * slot (col, val) pairs are broadcast with shuffles; B rows are gathered
//     as float4 through the read-only path, U slots in flight per lane;
//   * the row width W is a template parameter for W <= 32, so the fold /
//     group reduction and the C update positions are compile-time;
//   * C update (reading R11): rows whose source row has exactly one CELL row
//     are plain vector stores; the others (folded rows, P > 1) were zeroed by
//     zero_rows_kernel and receive red.global.add.v4.f32;
//   * rows of A with no CELL row are zeroed by zero_rows_kernel (R13).
#include "../lf_internal.cuh"

namespace lf {

namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kWarpsPerBlock = 8;

template <int VEC> struct Vec;
template <> struct Vec<4> {
    using T = float4;
    static __device__ __forceinline__ T zero() { return make_float4(0.f, 0.f, 0.f, 0.f); }
    static __device__ __forceinline__ T load(const float *p) { return __ldg(reinterpret_cast<const float4 *>(p)); }
    static __device__ __forceinline__ void fma(T &acc, float a, const T &b) {
        acc.x = fmaf(a, b.x, acc.x);
        acc.y = fmaf(a, b.y, acc.y);
        acc.z = fmaf(a, b.z, acc.z);
        acc.w = fmaf(a, b.w, acc.w);
    }
    static __device__ __forceinline__ void add_xor(T &acc, int o) {
        acc.x += __shfl_xor_sync(kFull, acc.x, o);
        acc.y += __shfl_xor_sync(kFull, acc.y, o);
        acc.z += __shfl_xor_sync(kFull, acc.z, o);
        acc.w += __shfl_xor_sync(kFull, acc.w, o);
    }
    static __device__ __forceinline__ void store(float *p, const T &v) {
        asm volatile("st.global.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w)
                     : "memory");
    }
    static __device__ __forceinline__ void red(float *p, const T &v) {
        asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
                     "f"(v.w)
                     : "memory");
    }
};
template <> struct Vec<1> {
    using T = float;
    static __device__ __forceinline__ T zero() { return 0.f; }
    static __device__ __forceinline__ T load(const float *p) { return __ldg(p); }
    static __device__ __forceinline__ void fma(T &acc, float a, const T &b) { acc = fmaf(a, b, acc); }
    static __device__ __forceinline__ void add_xor(T &acc, int o) { acc += __shfl_xor_sync(kFull, acc, o); }
    static __device__ __forceinline__ void store(float *p, const T &v) { *p = v; }
    static __device__ __forceinline__ void red(float *p, const T &v) { atomicAdd(p, v); }
};

// Lane layout for one J tile of JT = LPR * NV * VEC columns starting at j0.
template <int VEC, int G, int NV>
struct Layout {
    static constexpr int LPR = 32 / G;  // lanes per group
    static constexpr int JT = LPR * NV * VEC;
    static constexpr int U = (8 / NV) > 1 ? (8 / NV) : 2;  // slots in flight per lane
};

template <int VEC, int G, int NV>
struct Ctx {
    using V = Vec<VEC>;
    using VT = typename V::T;
    using L = Layout<VEC, G, NV>;
    const float *__restrict__ B;
    int64_t ldb;
    float *__restrict__ C;
    int64_t ldc;
    int J;
    int j0;
    int g, li;  // lane group, lane in group

    __device__ __forceinline__ int jcol(int m) const { return j0 + (m * L::LPR + li) * VEC; }
    __device__ __forceinline__ bool jok(int m) const { return jcol(m) < J; }

    // gather slot's B row slice (zero if padding)
    __device__ __forceinline__ void gather(int32_t c, VT (&b)[NV]) const {
#pragma unroll
        for (int m = 0; m < NV; m++) b[m] = (c >= 0 && jok(m)) ? V::load(B + (int64_t)c * ldb + jcol(m)) : V::zero();
    }
    __device__ __forceinline__ void write(int32_t tag, const VT (&acc)[NV]) const {
        if (tag < 0) return;
        float *row = C + (int64_t)(tag >> 1) * ldc;
#pragma unroll
        for (int m = 0; m < NV; m++) {
            if (!jok(m)) continue;
            if (tag & 1) V::red(row + jcol(m), acc[m]);
            else V::store(row + jcol(m), acc[m]);
        }
    }
};

// 32-slot task of a bucket with W = 2^T <= 32: 32/W CELL rows.
template <int VEC, int G, int NV, int T>
__device__ __forceinline__ void narrow_task(const Ctx<VEC, G, NV> &cx, int32_t c_l, float v_l, int32_t tag_l) {
    using C = Ctx<VEC, G, NV>;
    using V = typename C::V;
    using VT = typename C::VT;
    constexpr int W = 1 << T;
    constexpr int STEPS = 32 / G;                      // each step: one slot per group
    constexpr int RG = W >= G ? G : W;                 // groups sharing one CELL row
    constexpr int SPR = W >= G ? W / G : 1;            // steps per row
    constexpr int U = C::L::U < STEPS ? C::L::U : STEPS;
    constexpr int LPR = C::L::LPR;
    VT acc[NV];
#pragma unroll
    for (int m = 0; m < NV; m++) acc[m] = V::zero();
#pragma unroll
    for (int kb = 0; kb < STEPS; kb += U) {
        VT b[U][NV];
        float a[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
            const int slot = (kb + u) * G + cx.g;
            const int32_t c = __shfl_sync(kFull, c_l, slot);
            a[u] = __shfl_sync(kFull, v_l, slot);
            cx.gather(c, b[u]);
        }
#pragma unroll
        for (int u = 0; u < U; u++) {
            const int step = kb + u;
#pragma unroll
            for (int m = 0; m < NV; m++) V::fma(acc[m], a[u], b[u][m]);
            if ((step + 1) % SPR == 0) {  // a CELL row ends here (compile-time)
#pragma unroll
                for (int o = 1; o < RG; o <<= 1)
#pragma unroll
                    for (int m = 0; m < NV; m++) V::add_xor(acc[m], o * LPR);
                const int ro = (W >= G) ? step / SPR : step * (G / W) + cx.g / W;
                const int32_t tag = __shfl_sync(kFull, tag_l, ro);
                if (cx.g % RG == 0) cx.write(tag, acc);
#pragma unroll
                for (int m = 0; m < NV; m++) acc[m] = V::zero();
            }
        }
    }
}

// Accumulate n32 chunks of 32 slots starting at slot s0 (one CELL row / CSR
// row of arbitrary length n), then reduce over groups and write.
template <int VEC, int G, int NV>
__device__ __forceinline__ void wide_row(const Ctx<VEC, G, NV> &cx, const int32_t *__restrict__ col,
                                         const float *__restrict__ val, int64_t s0, int64_t n, int32_t tag,
                                         int lane) {
    using C = Ctx<VEC, G, NV>;
    using V = typename C::V;
    using VT = typename C::VT;
    constexpr int STEPS = 32 / G;
    constexpr int U = C::L::U < STEPS ? C::L::U : STEPS;
    VT acc[NV];
#pragma unroll
    for (int m = 0; m < NV; m++) acc[m] = V::zero();
    for (int64_t base = 0; base < n; base += 32) {
        const int64_t s = s0 + base + lane;
        const bool in = base + lane < n;
        const int32_t c_l = in ? __ldg(col + s) : -1;
        const float v_l = in ? __ldg(val + s) : 0.f;
        if (__ballot_sync(kFull, c_l >= 0) == 0) break;  // rest of the row is padding
#pragma unroll
        for (int kb = 0; kb < STEPS; kb += U) {
            VT b[U][NV];
            float a[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                const int slot = (kb + u) * G + cx.g;
                const int32_t c = __shfl_sync(kFull, c_l, slot);
                a[u] = __shfl_sync(kFull, v_l, slot);
                cx.gather(c, b[u]);
            }
#pragma unroll
            for (int u = 0; u < U; u++)
#pragma unroll
                for (int m = 0; m < NV; m++) V::fma(acc[m], a[u], b[u][m]);
        }
    }
#pragma unroll
    for (int o = 1; o < G; o <<= 1)
#pragma unroll
        for (int m = 0; m < NV; m++) V::add_xor(acc[m], o * C::L::LPR);
    if (cx.g == 0) cx.write(tag, acc);
}

template <int VEC, int G, int NV>
__global__ void __launch_bounds__(kWarpsPerBlock * 32) cell_spmm_kernel(SpmmArgs a) {
    using L = Layout<VEC, G, NV>;
    const int lane = threadIdx.x & 31;
    const int64_t gwarp = (int64_t)blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    const int64_t nwarps = (int64_t)gridDim.x * kWarpsPerBlock;
    Ctx<VEC, G, NV> cx{a.B, a.ldb, a.C, a.ldc, a.J, 0, lane / L::LPR, lane % L::LPR};
    int b = 0;
    for (int64_t task = gwarp; task < a.n_tasks; task += nwarps) {
        while (b + 1 < a.nb && a.buckets[b + 1].task_off <= task) b++;  // tasks ascend per warp
        const BucketDev bk = a.buckets[b];
        const int64_t tin = task - bk.task_off;
        if (bk.t > 5) {  // one CELL row of W = 2^t > 32 slots
            const int32_t tag = __ldg(a.row_tag + bk.row_off + tin);
            if (tag < 0) continue;
            for (int j0 = 0; j0 < a.J; j0 += L::JT) {
                cx.j0 = j0;
                wide_row<VEC, G, NV>(cx, a.col, a.val, bk.slot_off + tin * bk.task_slots, bk.task_slots, tag, lane);
            }
            continue;
        }
        const int64_t s0 = bk.slot_off + tin * 32;
        const int64_t ns = min((int64_t)32, bk.n_slots - tin * 32);
        const int32_t c_l = lane < ns ? __ldg(a.col + s0 + lane) : -1;
        const float v_l = lane < ns ? __ldg(a.val + s0 + lane) : 0.f;
        const int64_t nrows = ns >> bk.t;
        const int32_t tag_l = lane < nrows ? __ldg(a.row_tag + bk.row_off + ((tin * 32) >> bk.t) + lane) : -1;
        if (__ballot_sync(kFull, tag_l >= 0) == 0) continue;  // all padding
        for (int j0 = 0; j0 < a.J; j0 += L::JT) {
            cx.j0 = j0;
            switch (bk.t) {
            case 0: narrow_task<VEC, G, NV, 0>(cx, c_l, v_l, tag_l); break;
            case 1: narrow_task<VEC, G, NV, 1>(cx, c_l, v_l, tag_l); break;
            case 2: narrow_task<VEC, G, NV, 2>(cx, c_l, v_l, tag_l); break;
            case 3: narrow_task<VEC, G, NV, 3>(cx, c_l, v_l, tag_l); break;
            case 4: narrow_task<VEC, G, NV, 4>(cx, c_l, v_l, tag_l); break;
            default: narrow_task<VEC, G, NV, 5>(cx, c_l, v_l, tag_l); break;
            }
        }
    }
}

// Algorithm 1 on the GPU straight from CSR: one warp per row, same lane layout.
template <int VEC, int G, int NV>
__global__ void __launch_bounds__(kWarpsPerBlock * 32)
    csr_spmm_kernel(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col,
                    const float *__restrict__ val, int64_t n_rows, const float *__restrict__ B, int64_t ldb,
                    float *__restrict__ C, int64_t ldc, int J) {
    using L = Layout<VEC, G, NV>;
    const int lane = threadIdx.x & 31;
    const int64_t gwarp = (int64_t)blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    const int64_t nwarps = (int64_t)gridDim.x * kWarpsPerBlock;
    Ctx<VEC, G, NV> cx{B, ldb, C, ldc, J, 0, lane / L::LPR, lane % L::LPR};
    for (int64_t i = gwarp; i < n_rows; i += nwarps) {
        const int64_t rb = row_ptr[i], re = row_ptr[i + 1];
        for (int j0 = 0; j0 < J; j0 += L::JT) {
            cx.j0 = j0;
            wide_row<VEC, G, NV>(cx, col, val, rb, re - rb, (int32_t)(i << 1), lane);
        }
    }
}

// C rows whose source row has != 1 CELL rows: zero (empty rows are the
// result; multi-writer rows then receive red.add).  A warp scans 32 rows.
__global__ void zero_rows_kernel(const int32_t *__restrict__ row_cnt, int64_t n_rows, float *__restrict__ C,
                                 int64_t ldc, int J, int vec4) {
    const int lane = threadIdx.x & 31;
    const int64_t gwarp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t base = gwarp * 32; base < n_rows; base += nwarps * 32) {
        const int64_t i = base + lane;
        unsigned need = __ballot_sync(kFull, i < n_rows && __ldg(row_cnt + i) != 1);
        while (need) {
            const int src = __ffs(need) - 1;
            need &= need - 1;
            float *row = C + (base + src) * ldc;
            if (vec4) {
                for (int j = lane * 4; j < J; j += 128)
                    *reinterpret_cast<float4 *>(row + j) = make_float4(0.f, 0.f, 0.f, 0.f);
            } else {
                for (int j = lane; j < J; j += 32) row[j] = 0.f;
            }
        }
    }
}

template <int VEC, int G, int NV>
int blocks_for(const void *fn) {
    static int occ = 0, sms = 0;
    if (!occ) {
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, kWarpsPerBlock * 32, 0);
        if (occ <= 0) occ = 1;
        if (sms <= 0) sms = 148;
    }
    return occ * sms;
}

template <int VEC, int G, int NV>
cudaError_t run_cell(const SpmmArgs &a, cudaStream_t s) {
    auto fn = cell_spmm_kernel<VEC, G, NV>;
    int64_t want = (a.n_tasks + kWarpsPerBlock - 1) / kWarpsPerBlock;
    int grid = (int)std::max<int64_t>(1, std::min<int64_t>(want, blocks_for<VEC, G, NV>((const void *)fn)));
    fn<<<grid, kWarpsPerBlock * 32, 0, s>>>(a);
    return cudaGetLastError();
}

template <int VEC, int G, int NV>
cudaError_t run_csr(const lf_csr &A, const float *B, int64_t ldb, int J, float *C, int64_t ldc, cudaStream_t s) {
    auto fn = csr_spmm_kernel<VEC, G, NV>;
    int64_t want = (A.n_rows + kWarpsPerBlock - 1) / kWarpsPerBlock;
    int grid = (int)std::max<int64_t>(1, std::min<int64_t>(want, blocks_for<VEC, G, NV>((const void *)fn)));
    fn<<<grid, kWarpsPerBlock * 32, 0, s>>>(A.row_ptr, A.col_ind, A.val, A.n_rows, B, ldb, C, ldc, J);
    return cudaGetLastError();
}

bool vec4_ok(const float *B, int64_t ldb, const float *C, int64_t ldc, int J) {
    return J % 4 == 0 && ldb % 4 == 0 && ldc % 4 == 0 && ((uintptr_t)B & 15) == 0 && ((uintptr_t)C & 15) == 0;
}

}  // namespace

cudaError_t launch_zero_rows(const int32_t *row_cnt, int64_t n_rows, float *C, int64_t ldc, int J, cudaStream_t s) {
    if (n_rows == 0 || J == 0) return cudaSuccess;
    const int vec4 = (J % 4 == 0 && ldc % 4 == 0 && ((uintptr_t)C & 15) == 0) ? 1 : 0;
    int64_t warps = (n_rows + 31) / 32;
    int grid = (int)std::max<int64_t>(1, std::min<int64_t>((warps + 7) / 8, 148LL * 16));
    zero_rows_kernel<<<grid, 256, 0, s>>>(row_cnt, n_rows, C, ldc, J, vec4);
    return cudaGetLastError();
}

cudaError_t launch_cell_spmm(const SpmmArgs &a, cudaStream_t s) {
    if (a.n_tasks == 0 || a.J == 0) return cudaSuccess;
    if (vec4_ok(a.B, a.ldb, a.C, a.ldc, a.J)) {
        if (a.J <= 32) return run_cell<4, 4, 1>(a, s);
        if (a.J <= 64) return run_cell<4, 2, 1>(a, s);
        if (a.J <= 128) return run_cell<4, 1, 1>(a, s);
        if (a.J <= 256) return run_cell<4, 1, 2>(a, s);
        return run_cell<4, 1, 4>(a, s);
    }
    return run_cell<1, 1, 4>(a, s);
}

cudaError_t launch_csr_spmm(const lf_csr &A, const float *B, int64_t ldb, int J, float *C, int64_t ldc,
                            cudaStream_t s) {
    if (A.n_rows == 0 || J == 0) return cudaSuccess;
    if (vec4_ok(B, ldb, C, ldc, J)) {
        if (J <= 32) return run_csr<4, 4, 1>(A, B, ldb, J, C, ldc, s);
        if (J <= 64) return run_csr<4, 2, 1>(A, B, ldb, J, C, ldc, s);
        if (J <= 128) return run_csr<4, 1, 1>(A, B, ldb, J, C, ldc, s);
        if (J <= 256) return run_csr<4, 1, 2>(A, B, ldb, J, C, ldc, s);
        return run_csr<4, 1, 4>(A, B, ldb, J, C, ldc, s);
    }
    return run_csr<1, 1, 4>(A, B, ldb, J, C, ldc, s);
}

}  // namespace lf
