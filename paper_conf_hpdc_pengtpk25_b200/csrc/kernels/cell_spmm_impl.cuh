// cell_spmm_impl.cuh -- the CELL SpMM kernels (per-slot, grouped, mma.sync
// grouped) and their launch templates, shared by the translation units that
// instantiate them: cell_spmm.cu (dispatch, float4 / scalar per-slot
// kernels, CSR kernel), cell_spmm_v8.cu (256-bit per-slot kernels),
// cell_spmm_grp.cu (grouped and mma.sync kernels), cell_spmm_md.cu (the
// fused-row-exchange instantiations).  Split so nvcc compiles them in
// parallel.  Everything here has internal linkage.
#pragma once
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
#include "../lf_internal.cuh"

#include <algorithm>
#include <cstdio>
#include <vector>

namespace lf {

namespace {

constexpr unsigned kFull = 0xffffffffu;
constexpr int kWarpsPerBlock = 8;
#ifndef LF_SKIP_PAD
#define LF_SKIP_PAD 0  // measured: the per-slot predicate costs more than the skipped zero-row loads
#endif
#ifndef LF_ZERO_FIRST
#define LF_ZERO_FIRST 1  // empty rows zeroed before the gathers (overlapped), not in a tail phase
#endif
#ifndef LF_EPI_ZERO
#define LF_EPI_ZERO 1  // empty C rows zeroed in the SpMM kernel's epilogue
#endif
constexpr int kChunk = kWideChunk;  // consecutive tasks per warp per round
#ifndef LF_SPMM_MIN_BLOCKS
#define LF_SPMM_MIN_BLOCKS 4
#endif
constexpr int kMinBlocks = LF_SPMM_MIN_BLOCKS;  // resident 256-thread blocks per SM

__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ int32_t ld_stream(const int32_t *p, uint64_t pol) {
    int32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ float ld_stream(const float *p, uint64_t pol) {
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
    return v;
}

// Programmatic dependent launch: the SpMM kernel may start while
// zero_rows_kernel (launched just before it, writing only the rows that later
// receive red.add) is still running; a red waits for that grid first.
__device__ __forceinline__ void grid_dep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

template <int VEC> struct Vec;
template <> struct Vec<4> {
    using T = float4;
    static __device__ __forceinline__ T zero() { return make_float4(0.f, 0.f, 0.f, 0.f); }
#ifndef LF_BLOAD
#define LF_BLOAD 0  // B-row gathers: 0 = ld.global.nc; 1 = + L1::no_allocate; 2 = + L2 evict_last; 3 = L1 alloc + evict_last
#endif
    static __device__ __forceinline__ T load(const float *p) {
#if LF_BLOAD == 0
        return __ldg(reinterpret_cast<const float4 *>(p));
#else
        T v;
#if LF_BLOAD == 1
        asm("ld.global.nc.L1::no_allocate.v4.f32 {%0, %1, %2, %3}, [%4];"
            : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
#else
        uint64_t pl;
        asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
#if LF_BLOAD == 2
        asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
            : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pl));
#else
        asm("ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
            : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pl));
#endif
#endif
        return v;
#endif
    }
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
    // C row stores carry no "memory" clobber: C is only written by this
    // kernel (never read back), and a clobber would pin every later B-row
    // gather behind the store (no overlap of a row's write with the next
    // row's loads).  LF_ST_CLOBBER=1 restores it for measurement.
#ifndef LF_ST_CLOBBER
#define LF_ST_CLOBBER 0
#endif
    static __device__ __forceinline__ void store(float *p, const T &v, uint64_t pol) {
#if LF_ST_CLOBBER
        asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p),
                     "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "l"(pol)
                     : "memory");
#else
        asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p),
                     "f"(v.x), "f"(v.y), "f"(v.z), "f"(v.w), "l"(pol));
#endif
    }
    static __device__ __forceinline__ void red(float *p, const T &v) {
        grid_dep_wait();
        asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
                     "f"(v.w)
                     : "memory");
    }
};
// 8 floats per lane: one 256-bit load (ld.global.nc.v8.f32, sm_100) per B-row
// slice, half the gather instructions of float4 for the same row bytes
struct f8 {
    float4 a, b;
};
#ifndef LF_ST_V8
#define LF_ST_V8 1  // 256-bit C row stores (st.global.v8.f32): c2 0.585 -> 0.576 ms
#endif
template <> struct Vec<8> {
    using T = f8;
    static __device__ __forceinline__ T zero() { return {make_float4(0.f, 0.f, 0.f, 0.f), make_float4(0.f, 0.f, 0.f, 0.f)}; }
    static __device__ __forceinline__ T load(const float *p) {
        T v;
        asm("ld.global.nc.v8.f32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
            : "=f"(v.a.x), "=f"(v.a.y), "=f"(v.a.z), "=f"(v.a.w), "=f"(v.b.x), "=f"(v.b.y), "=f"(v.b.z), "=f"(v.b.w)
            : "l"(p));
        return v;
    }
    static __device__ __forceinline__ void fma(T &acc, float a, const T &b) {
        Vec<4>::fma(acc.a, a, b.a);
        Vec<4>::fma(acc.b, a, b.b);
    }
    static __device__ __forceinline__ void add_xor(T &acc, int o) {
        Vec<4>::add_xor(acc.a, o);
        Vec<4>::add_xor(acc.b, o);
    }
    static __device__ __forceinline__ void store(float *p, const T &v, uint64_t pol) {
#if LF_ST_V8
        asm volatile("st.global.L1::no_allocate.L2::cache_hint.v8.f32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8}, %9;" ::"l"(p),
                     "f"(v.a.x), "f"(v.a.y), "f"(v.a.z), "f"(v.a.w), "f"(v.b.x), "f"(v.b.y), "f"(v.b.z), "f"(v.b.w),
                     "l"(pol));
#else
        Vec<4>::store(p, v.a, pol);
        Vec<4>::store(p + 4, v.b, pol);
#endif
    }
    static __device__ __forceinline__ void red(float *p, const T &v) {
        Vec<4>::red(p, v.a);
        Vec<4>::red(p + 4, v.b);
    }
};
template <> struct Vec<1> {
    using T = float;
    static __device__ __forceinline__ T zero() { return 0.f; }
    static __device__ __forceinline__ T load(const float *p) { return __ldg(p); }
    static __device__ __forceinline__ void fma(T &acc, float a, const T &b) { acc = fmaf(a, b, acc); }
    static __device__ __forceinline__ void add_xor(T &acc, int o) { acc += __shfl_xor_sync(kFull, acc, o); }
    static __device__ __forceinline__ void store(float *p, const T &v, uint64_t) { *p = v; }
    static __device__ __forceinline__ void red(float *p, const T &v) {
        grid_dep_wait();
        atomicAdd(p, v);
    }
};

// tag helpers
__device__ __forceinline__ bool tag_whole(int32_t tag) { return (tag & 7) == 7; }  // S && F && L
__device__ __forceinline__ int32_t tag_row(int32_t tag) { return tag >> 3; }

#ifdef LF_TRACE
__device__ unsigned long long lf_trace_buf[2 * 148 * 64];
__device__ unsigned long long lf_trace_st[148 * 64];
__device__ unsigned int lf_trace_tasks[148 * 64];
__device__ unsigned long long lf_trace_t0;
#endif
// all-zero row that padding slots (colInd = -1, val = +0.0) gather from, so
// every slot issues the same unpredicated load (JT <= 512 floats)
__device__ float4 g_zero_row[128];

template <int VEC, int G, int NV>
struct Layout {
    static constexpr int LPR = 32 / G;  // lanes per group
    static constexpr int JT = LPR * NV * VEC;
#ifndef LF_U
#define LF_U 4
#endif
    static constexpr int U = (LF_U / NV) > 1 ? (LF_U / NV) : 2;  // slots in flight per lane
};

template <int VEC, int G, int NV, bool FULL, bool MD = false>
struct Ctx {
    using V = Vec<VEC>;
    using VT = typename V::T;
    using L = Layout<VEC, G, NV>;
    static constexpr int Gv = G, NVv = NV;
    const float *__restrict__ B;
    int64_t ldb;
    float *__restrict__ C;
    int64_t ldc;
    int J;
    int j0;
    int g, li;  // lane group, lane in group
    uint64_t pol;

    __device__ __forceinline__ int jcol(int m) const { return j0 + (m * L::LPR + li) * VEC; }
    __device__ __forceinline__ bool jok(int m) const { return FULL || jcol(m) < J; }

    // address of B row c, or of the zero row for a padding slot (computed once
    // per slot when a chunk is resolved, not in the gather loop)
    __device__ __forceinline__ const float *rowaddr(int32_t c) const {
        return c >= 0 ? B + (int64_t)c * ldb : reinterpret_cast<const float *>(g_zero_row) - j0;
    }
    __device__ __forceinline__ void gather(const float *r, VT (&b)[NV]) const {
#if LF_SKIP_PAD
        // a padding slot (zero-row address) issues no load at all
        const bool real = r != reinterpret_cast<const float *>(g_zero_row) - j0;
#else
        const bool real = true;
#endif
#pragma unroll
        for (int m = 0; m < NV; m++) b[m] = (jok(m) && real) ? V::load(r + jcol(m)) : V::zero();
    }
    // write one C row slice: plain store when this write is the row's only one
    __device__ __forceinline__ void write_to(float *p, bool plain, const VT (&acc)[NV]) const {
#pragma unroll
        for (int m = 0; m < NV; m++) {
            if (!jok(m)) continue;
#ifdef LF_DIAG_NOWRITE  // diagnostic builds only: drop the C traffic
            if (reinterpret_cast<const float *>(&acc[m])[0] != 1234.5f) continue;
#endif
            if (plain) V::store(p + jcol(m), acc[m], pol);
            else V::red(p + jcol(m), acc[m]);
        }
    }
    // write one C row slice (plain store when this write is the row's only
    // one); with a fused row exchange (a.n_dst > 0, lf_spmm_ex) the same slice
    // goes to every destination C (local and peers) straight from the
    // registers.  The destinations are read from the kernel parameters, not
    // kept in registers.
    // (MD: the kernel instantiation for lf_spmm_ex with destinations; the
    // plain instantiation carries no trace of it -- a runtime test there cost
    // the grouped kernel 4%)
    __device__ __forceinline__ void write(const SpmmArgs &a, int32_t row, bool plain, const VT (&acc)[NV]) const {
        if constexpr (MD) {
            for (int d = 0; d < a.n_dst; d++) write_to(ld_dst(a.dst, d) + (a.row_base + row) * ldc, plain, acc);
        } else {
            write_to(C + (int64_t)row * ldc, plain, acc);
        }
    }
    __device__ __forceinline__ void write(int32_t row, bool plain, const VT (&acc)[NV]) const {
        write_to(C + (int64_t)row * ldc, plain, acc);
    }
    __device__ __forceinline__ void zero(VT (&acc)[NV]) const {
#pragma unroll
        for (int m = 0; m < NV; m++) acc[m] = V::zero();
    }
    // sum the G lane groups (all hold partial sums of the same row)
    __device__ __forceinline__ void reduce_groups(VT (&acc)[NV]) const {
#pragma unroll
        for (int o = 1; o < G; o <<= 1)
#pragma unroll
            for (int m = 0; m < NV; m++) V::add_xor(acc[m], o * L::LPR);
    }
};

// The current 32-slot chunk is RESOLVED in shared memory per warp: every
// slot's B-row address (zero row for padding) and value, ordered so that lane
// group g finds its steps k, k+1 (slots k*G+g, (k+1)*G+g) adjacent -- one
// broadcast LDS.128 + one LDS.64 feed two gathers.
struct Resolved {
    const float *addr[32];
    float val[32];
};

template <int G>
__device__ __forceinline__ int stage_pos(int s) { return (s % G) * (32 / G) + s / G; }

// synchronous path: (c, v) of the lane's slot from registers
template <int G, class Cx>
__device__ __forceinline__ void stage(const Cx &cx, Resolved &r, int lane, int32_t c, float v) {
    __syncwarp();
    const int p = stage_pos<G>(lane);
    r.addr[p] = cx.rowaddr(c);
    r.val[p] = v;
    __syncwarp();
}

// asynchronous path: raw (c, v bits) already landed at stage positions
template <class Cx>
__device__ __forceinline__ void resolve(const Cx &cx, const int2 *raw, Resolved &r, int lane) {
    const int2 e = raw[lane];
    r.addr[lane] = cx.rowaddr(e.x);
    r.val[lane] = __int_as_float(e.y);
    __syncwarp();
}

template <class Cx, int U>
__device__ __forceinline__ void fetch(const Cx &cx, const Resolved &r, int kb, typename Cx::VT (&b)[U][Cx::NVv],
                                      float (&a)[U]) {
#pragma unroll
    for (int u = 0; u < U; u += 2) {
        const int p = cx.g * (32 / Cx::Gv) + kb + u;
        const ulonglong2 ad = *reinterpret_cast<const ulonglong2 *>(&r.addr[p]);
        const float2 vv = *reinterpret_cast<const float2 *>(&r.val[p]);
        a[u] = vv.x;
        cx.gather(reinterpret_cast<const float *>(ad.x), b[u]);
        a[u + 1] = vv.y;
        cx.gather(reinterpret_cast<const float *>(ad.y), b[u + 1]);
    }
}

// the staged 32 slots accumulated into acc, no row boundary; slots at and
// beyond n_real (a warp-uniform count: padding is a suffix of a CELL row)
// are skipped a batch at a time
template <class Cx>
__device__ __forceinline__ void accum32(const Cx &cx, const Resolved &sw, typename Cx::VT (&acc)[Cx::NVv],
                                        int n_real = 32) {
    using V = typename Cx::V;
    using VT = typename Cx::VT;
    constexpr int NV = Cx::NVv;
    constexpr int STEPS = 32 / Cx::Gv;
    constexpr int U = Cx::L::U < STEPS ? Cx::L::U : STEPS;
#pragma unroll
    for (int kb = 0; kb < STEPS; kb += U) {
        if (kb * Cx::Gv >= n_real) break;
        VT b[U][NV];
        float a[U];
        fetch<Cx, U>(cx, sw, kb, b, a);
#pragma unroll
        for (int u = 0; u < U; u++)
#pragma unroll
            for (int m = 0; m < NV; m++) V::fma(acc[m], a[u], b[u][m]);
    }
}

// 32-slot task of a bucket with W = 2^T < 32: 32/W CELL rows, each written.
template <class Cx, int T>
__device__ __forceinline__ void narrow_task(const SpmmArgs &args, const Cx &cx, const Resolved &sw, int32_t tag_l) {
    using V = typename Cx::V;
    using VT = typename Cx::VT;
    constexpr int NV = Cx::NVv, G = Cx::Gv;
    constexpr int W = 1 << T;
    constexpr int STEPS = 32 / G;            // each step: one slot per group
    constexpr int RG = W >= G ? G : W;       // groups sharing one CELL row
    constexpr int SPR = W >= G ? W / G : 1;  // steps per row
    constexpr int U = Cx::L::U < STEPS ? Cx::L::U : STEPS;
    constexpr int LPR = Cx::L::LPR;
    VT acc[NV];
    cx.zero(acc);
#pragma unroll
    for (int kb = 0; kb < STEPS; kb += U) {
        VT b[U][NV];
        float a[U];
        fetch<Cx, U>(cx, sw, kb, b, a);
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
                if (cx.g % RG == 0 && tag >= 0) cx.write(args, tag_row(tag), tag_whole(tag), acc);
                cx.zero(acc);
            }
        }
    }
}

// Zero the C rows whose mode is in mode_mask (bit per kRow* value): the
// rows that receive red.global.add must hold +0.0 first.  A warp scans 32 rows.
__device__ __forceinline__ void zero_row(float *row, int J, int lane, bool vec4, uint64_t pol) {
    if (vec4) {
        for (int j = lane * 4; j < J; j += 128) Vec<4>::store(row + j, make_float4(0.f, 0.f, 0.f, 0.f), pol);
    } else {
        for (int j = lane; j < J; j += 32) row[j] = 0.f;
    }
}

__device__ __forceinline__ void zero_rows_warp(const uint8_t *__restrict__ row_mode, int64_t n_rows, float *C,
                                               int64_t ldc, int J, bool vec4, unsigned mode_mask, int64_t wid,
                                               int64_t nw, int lane, uint64_t pol, int nd = 0,
                                               float *const *dp = nullptr, int64_t rb = 0) {
    for (int64_t base = wid * 32; base < n_rows; base += nw * 32) {
        const int64_t i = base + lane;
        unsigned need = __ballot_sync(kFull, i < n_rows && ((mode_mask >> __ldg(row_mode + i)) & 1u));
        while (need) {
            const int src = __ffs(need) - 1;
            need &= need - 1;
            if (nd == 0) zero_row(C + (base + src) * ldc, J, lane, vec4, pol);
            for (int d = 0; d < nd; d++) zero_row(ld_dst(dp, d) + (rb + base + src) * ldc, J, lane, vec4, pol);
        }
    }
}

// ---- asynchronous staging ----------------------------------------------
// A warp owns two stage buffers; while it gathers B rows for the slots in
// one, cp.async (LDGSTS, L2 evict_first) fills the other with the next
// 32 slots (and their row tags), so the index/value stream never waits in
// registers.
struct WarpStage {
    int2 slot[2][32];   // raw (col, val bits) at stage_pos order, filled by cp.async
    int32_t tag[2][32]; // row tags of the staged slots' rows
    Resolved res;       // the chunk being gathered
};

__device__ __forceinline__ void cp_async4(void *dst, const void *src, uint64_t pol) {
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 4, %2;" ::"r"(
                     (uint32_t)__cvta_generic_to_shared(dst)),
                 "l"(src), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }

// ---- dynamic work queues --------------------------------------------------
// Warps claim ranges of tasks with atomicAdd on per-launch counters (ctr[0]:
// wide class, ctr[1]: narrow class).  Guided sizes: kChunk tasks while much
// work remains, shrinking to 1 near the end so the last claims are short.  A
// claim is issued one range ahead and read (shuffle from lane 0) only when
// the warp moves on, so the atomic's latency is hidden; claims grow per warp,
// so bucket cursors only move forward.
__device__ __forceinline__ int claim_size(int64_t n, int64_t hint, int64_t nw, int chunk = kChunk) {
    const int64_t left = n - hint;
    return (int)max((int64_t)1, min((int64_t)chunk, left / (2 * nw)));
}
#ifndef LF_GROUP_CHUNK
#define LF_GROUP_CHUNK 8  // groups per claim on the grouped path
#endif
__device__ __forceinline__ unsigned long long claim_issue(unsigned long long *ctr, int size, int lane) {
    return lane == 0 ? atomicAdd(ctr, (unsigned long long)size) : 0ull;
}
__device__ __forceinline__ int64_t claim_get(unsigned long long raw) {
    return (int64_t)__shfl_sync(kFull, raw, 0);
}

// W < 32 class: a task is 32 slots = 32/W rows of one bucket.  Returns t.
template <int G>
__device__ __forceinline__ int issue_narrow(const SpmmArgs &a, int64_t task, int &bcur, int lane, uint64_t pol,
                                            WarpStage &st, int buf) {
    while (bcur + 1 < a.nb_n && __ldg(&a.bk_n[bcur + 1].task_off) <= task) bcur++;
    const BucketDev *bk = a.bk_n + bcur;
    const int64_t tin = task - __ldg(&bk->task_off);
    const int t = __ldg(&bk->t);
    const int64_t s0 = __ldg(&bk->slot_off) + tin * 32;
    const int64_t ns = min((int64_t)32, __ldg(&bk->n_slots) - tin * 32);
    const int64_t nrows = ns >> t;
    int2 *dst = &st.slot[buf][stage_pos<G>(lane)];
    if (lane < ns) {
        cp_async4(&dst->x, a.col + s0 + lane, pol);
        cp_async4(&dst->y, a.val + s0 + lane, pol);
    } else {
        *dst = make_int2(-1, 0);
    }
    if (lane < nrows) cp_async4(&st.tag[buf][lane], a.row_tag + __ldg(&bk->row_off) + ((tin * 32) >> t) + lane, pol);
    else st.tag[buf][lane] = -1;
    cp_commit();
    return t;
}

template <class Cx>
__device__ __forceinline__ void narrow_loop(const SpmmArgs &a, const Cx &cx0, WarpStage &st, int lane, int64_t nw,
                                            uint64_t pol) {
    constexpr int G = Cx::Gv, JT = Cx::L::JT;
    Cx cx = cx0;
    const int64_t n = a.n_tasks_n;
    int sz = claim_size(n, 0, nw);
    int64_t task = claim_get(claim_issue(a.ctr + 1, sz, lane));
    if (task >= n) return;
    int64_t tend = min(task + sz, n);
    int sz2 = claim_size(n, task, nw);
    unsigned long long raw = claim_issue(a.ctr + 1, sz2, lane);
    int bcur = 0, buf = 0;
    int t = issue_narrow<G>(a, task, bcur, lane, pol, st, 0);
    while (task < n) {
        int64_t tn = task + 1;
        if (tn >= tend) {
            tn = min(claim_get(raw), n);
            tend = min(tn + sz2, n);
            sz2 = claim_size(n, tn, nw);
            raw = claim_issue(a.ctr + 1, sz2, lane);
        }
        int tnext = 0;
        if (tn < n) tnext = issue_narrow<G>(a, tn, bcur, lane, pol, st, buf ^ 1);
        else cp_commit();
        cp_wait1();
        __syncwarp();
        const int32_t tag_l = st.tag[buf][lane];
        if (__ballot_sync(kFull, tag_l >= 0)) {
            const Resolved &sw = st.res;
            for (int j0 = 0; j0 < a.J; j0 += JT) {
                cx.j0 = j0;
                resolve(cx, st.slot[buf], st.res, lane);
                switch (t) {
                case 0: narrow_task<Cx, 0>(a, cx, sw, tag_l); break;
                case 1: narrow_task<Cx, 1>(a, cx, sw, tag_l); break;
                case 2: narrow_task<Cx, 2>(a, cx, sw, tag_l); break;
                case 3: narrow_task<Cx, 3>(a, cx, sw, tag_l); break;
                default: narrow_task<Cx, 4>(a, cx, sw, tag_l); break;
                }
            }
        }
        __syncwarp();
        buf ^= 1;
        task = tn;
        t = tnext;
    }
}

// W >= 32 class: a task is one CELL row = W/32 chunks of 32 slots.
struct WideCursor {
    int64_t task;
    int k, nch;  // 32-slot piece within the row, pieces per row
    int last;    // task is the last of its warp chunk (flush pending runs after it)
};

template <int G>
__device__ __forceinline__ void issue_wide(const SpmmArgs &a, const WideCursor &c, int bcur, int lane,
                                           uint64_t pol, WarpStage &st, int buf) {
    const BucketDev *bk = a.bk_w + bcur;
    const int64_t tin = c.task - __ldg(&bk->task_off);
    const int pl = __ldg(&bk->piece_log2);  // task = piece (tin & (2^pl - 1)) of CELL row tin >> pl
    const int64_t s = __ldg(&bk->slot_off) + ((tin >> pl) << __ldg(&bk->t)) + ((tin & ((1 << pl) - 1)) << kPieceLog2) +
                      32 * c.k + lane;
    int2 *dst = &st.slot[buf][stage_pos<G>(lane)];
    cp_async4(&dst->x, a.col + s, pol);
    cp_async4(&dst->y, a.val + s, pol);
    if (c.k == 0 && lane == 0) cp_async4(&st.tag[buf][0], a.row_tag + __ldg(&bk->row_off) + (tin >> pl), pol);
    cp_commit();
}

__device__ __forceinline__ int wide_nch(const SpmmArgs &a, int64_t task, int &bcur) {
    while (bcur + 1 < a.nb_w && __ldg(&a.bk_w[bcur + 1].task_off) <= task) bcur++;
    return 1 << (min(__ldg(&a.bk_w[bcur].t), kPieceLog2) - 5);
}

// Run-aligned claims: a claimed range [x, x + size) of the wide class really
// covers [bound(x), bound(x + size)) with bound(x) = x + run_bound[x]
// (run_bounds_kernel), so a whole run -- all CELL rows of a folded source
// row, <= kMaxRun -- never straddles two warps and is one plain store.
__device__ __forceinline__ int64_t chunk_bound(const SpmmArgs &a, int64_t x) {
    return x >= a.n_tasks_w ? a.n_tasks_w : min(a.n_tasks_w, x + (int64_t)__ldg(a.run_bound + x));
}

template <class Cx>
__device__ __forceinline__ void wide_loop(const SpmmArgs &a, const Cx &cx, WarpStage &st, int lane, int64_t nw,
                                          uint64_t pol) {
    using VT = typename Cx::VT;
    constexpr int NV = Cx::NVv, G = Cx::Gv;
    const int64_t n = a.n_tasks_w;
    // current range [rs, re); next claimed range (x1, sz1) with its bounds
    // loaded one range ahead; the claim after it in flight (raw, sz2)
    int sz0 = claim_size(n, 0, nw);
    int64_t x0 = claim_get(claim_issue(a.ctr, sz0, lane));
    if (x0 >= n) return;
    int sz1 = claim_size(n, x0, nw);
    int64_t x1 = claim_get(claim_issue(a.ctr, sz1, lane));
    int sz2 = claim_size(n, x1, nw);
    unsigned long long raw = claim_issue(a.ctr, sz2, lane);
    int64_t rs = chunk_bound(a, x0), re = chunk_bound(a, x0 + sz0);
    int64_t nrs = chunk_bound(a, x1), nre = chunk_bound(a, x1 + sz1);
    while (rs >= re && x0 < n) {  // empty range: its tasks belong to the previous range's run
        x0 = x1;
        rs = nrs;
        re = nre;
        x1 = claim_get(raw);
        sz1 = sz2;
        sz2 = claim_size(n, x1, nw);
        raw = claim_issue(a.ctr, sz2, lane);
        nrs = chunk_bound(a, x1);
        nre = chunk_bound(a, x1 + sz1);
    }
    if (x0 >= n) return;
    int bcur = 0, buf = 0;
    WideCursor cur{rs, 0, 0, 0};
    cur.nch = wide_nch(a, cur.task, bcur);
    int bcur_cur = bcur;
    issue_wide<G>(a, cur, bcur, lane, pol, st, 0);
    VT acc[NV];
    cx.zero(acc);
    int32_t pend = -1;     // tag of the run accumulated in acc (-1: none)
    int32_t row_tag = -1;  // tag of the row being streamed
    bool run_first = false;
    while (cur.task < n) {
        // successor piece: next 32 slots of the row, next task, or the first
        // task of the warp's next non-empty chunk
        WideCursor nx = cur;
        if (cur.k + 1 < cur.nch) {
            nx.k = cur.k + 1;
        } else {
            nx.k = 0;
            nx.task = cur.task + 1;
            if (nx.task >= re) {
                cur.last = 1;
                do {
                    x0 = x1;
                    rs = nrs;
                    re = nre;
                    x1 = claim_get(raw);
                    sz1 = sz2;
                    sz2 = claim_size(n, x1, nw);
                    raw = claim_issue(a.ctr, sz2, lane);
                    nrs = chunk_bound(a, x1);
                    nre = chunk_bound(a, x1 + sz1);
                } while (rs >= re && x0 < n);
                nx.task = x0 < n ? rs : n;
            }
        }
        int bcur_nx = bcur_cur;
        if (nx.task < n) {
            if (nx.k == 0) {
                nx.nch = wide_nch(a, nx.task, bcur);
                bcur_nx = bcur;
            }
            issue_wide<G>(a, nx, bcur_nx, lane, pol, st, buf ^ 1);
        } else {
            cp_commit();
        }
        cp_wait1();
        __syncwarp();
        if (cur.k == 0) {
            row_tag = st.tag[buf][0];
            if (row_tag >= 0) {
                if (pend >= 0 && tag_row(pend) != tag_row(row_tag)) {  // previous run split off: red
                    cx.reduce_groups(acc);
                    if (cx.g == 0) cx.write(a, tag_row(pend), false, acc);
                    cx.zero(acc);
                    pend = -1;
                }
                if (pend < 0) run_first = (row_tag & 2) != 0;
            }
        }
        const int n_real = row_tag >= 0 ? __popc(__ballot_sync(kFull, st.slot[buf][stage_pos<G>(lane)].x >= 0)) : 0;
        if (n_real > 0) {
            resolve(cx, st.slot[buf], st.res, lane);
            accum32(cx, st.res, acc, n_real);
        }
        if (cur.k == cur.nch - 1) {
#ifdef LF_TRACE
            if (lane == 0) lf_trace_tasks[blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5)]++;
#endif
            if (row_tag >= 0) {
                pend = row_tag;
                if (row_tag & 1) {  // last sub-row of the segment completes the run
                    cx.reduce_groups(acc);
                    if (cx.g == 0) cx.write(a, tag_row(row_tag), run_first && (row_tag & 4), acc);
                    cx.zero(acc);
                    pend = -1;
                }
            }
            if (cur.last && pend >= 0) {
                cx.reduce_groups(acc);
                if (cx.g == 0) cx.write(a, tag_row(pend), false, acc);
                cx.zero(acc);
                pend = -1;
            }
        }
        __syncwarp();
        buf ^= 1;
        cur = nx;
        bcur_cur = bcur_nx;
    }
}

// J wider than one pass (J > JT): each row is streamed once per J tile,
// synchronously, and every tile writes its slice (no run merging).
template <class Cx>
__device__ __forceinline__ void wide_loop_tiled(const SpmmArgs &a, const Cx &cx0, WarpStage &st, int lane,
                                                uint64_t pol) {
    using VT = typename Cx::VT;
    constexpr int NV = Cx::NVv, G = Cx::Gv, JT = Cx::L::JT;
    Cx cx = cx0;
    int bcur = 0;
    for (int64_t c = claim_get(claim_issue(a.ctr, kChunk, lane)); c < a.n_tasks_w;
         c = claim_get(claim_issue(a.ctr, kChunk, lane))) {
        for (int64_t task = c; task < min(c + kChunk, a.n_tasks_w); task++) {
            const int nch = wide_nch(a, task, bcur);
            const BucketDev *bk = a.bk_w + bcur;
            const int64_t tin = task - __ldg(&bk->task_off);
            const int pl = __ldg(&bk->piece_log2);
            const int32_t tag = __ldg(a.row_tag + __ldg(&bk->row_off) + (tin >> pl));
            if (tag < 0) continue;
            const int64_t s0 = __ldg(&bk->slot_off) + ((tin >> pl) << __ldg(&bk->t)) +
                               ((tin & ((1 << pl) - 1)) << kPieceLog2);
            for (int j0 = 0; j0 < a.J; j0 += JT) {
                cx.j0 = j0;
                VT acc[NV];
                cx.zero(acc);
                for (int k = 0; k < nch; k++) {
                    const int32_t c_l = ld_stream(a.col + s0 + 32 * k + lane, pol);
                    const float v_l = ld_stream(a.val + s0 + 32 * k + lane, pol);
                    if (__ballot_sync(kFull, c_l >= 0) == 0) break;  // rest is padding
                    stage<G>(cx, st.res, lane, c_l, v_l);
                    accum32(cx, st.res, acc);
                }
                cx.reduce_groups(acc);
                if (cx.g == 0) cx.write(a, tag_row(tag), tag_whole(tag), acc);
            }
        }
    }
}

// Blocks [0, a.blocks_n) start on the W < 32 queue, the others on the
// W >= 32 queue; a warp whose queue is drained helps with the other one.
// The two loops run one after the other (no live state in common), so each
// is register-allocated alone.  Epilogue: empty C rows are zeroed.
// resident blocks per SM: wider J slices per lane (NV float4) need more
// registers for the accumulators and the gathers in flight (no spills)
#ifndef LF_V8_MIN_BLOCKS
#define LF_V8_MIN_BLOCKS 3  // 8 floats per lane (80 registers)
#endif
constexpr int min_blocks(int NV, int VEC = 4) {
    return NV * VEC >= 16 ? 2 : NV * VEC == 8 ? LF_V8_MIN_BLOCKS : kMinBlocks;
}

template <int VEC, int G, int NV, bool FULL, bool MD = false>
__global__ void __launch_bounds__(kWarpsPerBlock * 32, min_blocks(NV, VEC)) cell_spmm_kernel(const SpmmArgs a) {
    using Cx = Ctx<VEC, G, NV, FULL, MD>;
    using L = Layout<VEC, G, NV>;
    __shared__ __align__(16) WarpStage stage_buf[kWarpsPerBlock];
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    WarpStage &st = stage_buf[w];
    const uint64_t pol = policy_evict_first();
    const Cx cx{a.B, a.ldb, a.C, a.ldc, a.J, 0, lane / L::LPR, lane % L::LPR, pol};
    const bool tiled = a.J > L::JT;
#ifdef LF_TRACE
    {
        unsigned long long t0;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        if (lane == 0) { lf_trace_st[blockIdx.x * kWarpsPerBlock + w] = t0; lf_trace_tasks[blockIdx.x * kWarpsPerBlock + w] = 0; }
    }
#endif
    const int64_t nw = (int64_t)gridDim.x * kWarpsPerBlock;
#ifdef LF_DIAG_NOWRITE
    constexpr bool kZero = false;
#else
    constexpr bool kZero = LF_EPI_ZERO;
#endif
    // rows of A with no CELL row are written +0.0 (R13) by every warp for its
    // share of the rows; done first, the write traffic overlaps the gathers
    // of the warps already streaming instead of forming a tail phase
    if (kZero && LF_ZERO_FIRST)
        zero_rows_warp(a.row_mode, a.n_rows, a.C, a.ldc, a.J, VEC >= 4, 1u << kRowEmpty,
                       (int64_t)blockIdx.x * kWarpsPerBlock + w, nw, lane, pol, MD ? a.n_dst : 0, a.dst, a.row_base);
    if ((int)blockIdx.x < a.blocks_n) {
        narrow_loop(a, cx, st, lane, nw, pol);
        if (tiled) wide_loop_tiled(a, cx, st, lane, pol);
        else wide_loop(a, cx, st, lane, nw, pol);
    } else {
        if (tiled) wide_loop_tiled(a, cx, st, lane, pol);
        else wide_loop(a, cx, st, lane, nw, pol);
        narrow_loop(a, cx, st, lane, nw, pol);
    }
#ifdef LF_TRACE
    unsigned long long t_work;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_work));
#endif
    if (kZero && !LF_ZERO_FIRST)
        zero_rows_warp(a.row_mode, a.n_rows, a.C, a.ldc, a.J, VEC >= 4, 1u << kRowEmpty,
                       (int64_t)blockIdx.x * kWarpsPerBlock + w, (int64_t)gridDim.x * kWarpsPerBlock, lane, pol,
                       MD ? a.n_dst : 0, a.dst, a.row_base);
    // the last warp out resets the queue counters for the next launch that
    // uses this slot (every claim of every warp is ordered before its fence)
    if (lane == 0) {
        __threadfence();
        if (atomicAdd(a.ctr + 2, 1ull) == (unsigned long long)gridDim.x * kWarpsPerBlock - 1) {
            __threadfence();
            a.ctr[0] = 0;
            a.ctr[1] = 0;
            a.ctr[2] = 0;
        }
    }
#ifdef LF_TRACE
    if (lane == 0) lf_trace_buf[(blockIdx.x * kWarpsPerBlock + w) * 2] = t_work;
    unsigned long long t_end;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_end));
    if (lane == 0) lf_trace_buf[(blockIdx.x * kWarpsPerBlock + w) * 2 + 1] = t_end;
#endif
}

// Algorithm 1 on the GPU straight from CSR: one warp per row, same lane layout.
template <int VEC, int G, int NV, bool FULL>
__global__ void __launch_bounds__(kWarpsPerBlock * 32)
    csr_spmm_kernel(const int64_t *__restrict__ row_ptr, const int32_t *__restrict__ col,
                    const float *__restrict__ val, int64_t n_rows, const float *__restrict__ B, int64_t ldb,
                    float *__restrict__ C, int64_t ldc, int J) {
    using Cx = Ctx<VEC, G, NV, FULL>;
    using VT = typename Cx::VT;
    using L = Layout<VEC, G, NV>;
    __shared__ __align__(16) Resolved stage_buf[kWarpsPerBlock];
    const int lane = threadIdx.x & 31;
    Resolved &sw = stage_buf[threadIdx.x >> 5];
    const int64_t gwarp = (int64_t)blockIdx.x * kWarpsPerBlock + (threadIdx.x >> 5);
    const int64_t nwarps = (int64_t)gridDim.x * kWarpsPerBlock;
    const uint64_t pol = policy_evict_first();
    Cx cx{B, ldb, C, ldc, J, 0, lane / L::LPR, lane % L::LPR, pol};
    for (int64_t i = gwarp; i < n_rows; i += nwarps) {
        const int64_t rb = row_ptr[i], re = row_ptr[i + 1];
        for (int j0 = 0; j0 < J; j0 += L::JT) {
            cx.j0 = j0;
            VT acc[NV];
            cx.zero(acc);
            for (int64_t base = rb; base < re; base += 32) {
                const bool in = base + lane < re;
                stage<G>(cx, sw, lane, in ? ld_stream(col + base + lane, pol) : -1,
                         in ? ld_stream(val + base + lane, pol) : 0.f);
                accum32(cx, sw, acc);
            }
            cx.reduce_groups(acc);
            if (cx.g == 0) cx.write((int32_t)i, true, acc);
        }
    }
}

__global__ void zero_rows_kernel(const uint8_t *__restrict__ row_mode, int64_t n_rows, float *__restrict__ C,
                                 int64_t ldc, int J, int vec4, unsigned mode_mask, int nd, float *const *dp,
                                 int64_t rb) {
    asm volatile("griddepcontrol.launch_dependents;");
    const int lane = threadIdx.x & 31;
    const int64_t gwarp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    zero_rows_warp(row_mode, n_rows, C, ldc, J, vec4 != 0, mode_mask, gwarp, nwarps, lane,
                   policy_evict_first(), nd, dp, rb);
}

#ifndef LF_CARVEOUT
#define LF_CARVEOUT -1  // >= 0: preferred shared-memory carveout (percent of the unified L1/smem) of the SpMM kernels
#endif
template <typename F>
int resident_blocks(F fn) {
    int occ = 0;
    const int sms = sm_count();
    if (LF_CARVEOUT >= 0) cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, LF_CARVEOUT);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, kWarpsPerBlock * 32, 0);
#ifndef LF_SPMM_GRID_BPS
#define LF_SPMM_GRID_BPS 0  // > 0: SpMM grids hold at most this many blocks per SM (the rest of the SM is left to
                            // kernels of other streams, e.g. the next step's configure / build)
#endif
    if (LF_SPMM_GRID_BPS > 0) occ = std::min(occ, LF_SPMM_GRID_BPS);
    return std::max(1, occ) * std::max(1, sms);
}

template <int VEC, int G, int NV, bool FULL, bool MD = false>
cudaError_t run_cell(const SpmmArgs &a0, cudaStream_t s) {
    static int caps[64];
    auto fn = cell_spmm_kernel<VEC, G, NV, FULL, MD>;
    int &cap = caps[current_device()];
    if (!cap) cap = resident_blocks(fn);
    SpmmArgs a = a0;
    const int64_t per_block = kWarpsPerBlock * kChunk;
    const int64_t want_n = (a.n_tasks_n + per_block - 1) / per_block;
    const int64_t want_w = (a.n_tasks_w + per_block - 1) / per_block;
    // split the resident blocks in proportion to the slots of each class
    const double frac_n = a.slots_n + a.slots_w > 0 ? (double)a.slots_n / (double)(a.slots_n + a.slots_w) : 0.0;
    int64_t bn = want_n ? std::max<int64_t>(1, (int64_t)(frac_n * cap + 0.5)) : 0;
    int64_t bw = want_w ? std::max<int64_t>(1, cap - bn) : 0;
    bn = std::min(bn, want_n);
    bw = std::min(bw, want_w);
    a.blocks_n = (int)bn;
    // enough blocks for the empty-row epilogue even without tasks
    const int64_t want_z = std::min<int64_t>(cap, (a.n_rows + 32 * kWarpsPerBlock - 1) / (32 * kWarpsPerBlock));
    const int grid = (int)std::max<int64_t>(bn + bw, want_z);
    if (grid == 0) return cudaSuccess;
    // a.ctr: the handle's counter slot for this launch (zero; reset by the
    // kernel's last warp)
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(kWarpsPerBlock * 32);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;  // overlap zero_rows_kernel
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, fn, a);
    if (e != cudaSuccess) return e;
#ifdef LF_TRACE
    {
        static std::vector<unsigned long long> h(2 * 148 * 64);
        cudaStreamSynchronize(s);
        cudaMemcpyFromSymbol(h.data(), lf_trace_buf, h.size() * 8);
        static std::vector<unsigned long long> hs(148 * 64);
        static std::vector<unsigned int> ht(148 * 64);
        cudaMemcpyFromSymbol(hs.data(), lf_trace_st, hs.size() * 8);
        cudaMemcpyFromSymbol(ht.data(), lf_trace_tasks, ht.size() * 4);
        const int nw = grid * kWarpsPerBlock;
        unsigned long long mn = ~0ull, mx = 0;
        for (int i = 0; i < nw; i++) { mn = std::min(mn, hs[i]); mx = std::max(mx, h[2 * i + 1]); }
        {
            std::vector<unsigned> tt(ht.begin() + a.blocks_n * kWarpsPerBlock, ht.begin() + nw);
            std::sort(tt.begin(), tt.end());
            std::vector<double> st0;
            for (int i = 0; i < nw; i++) st0.push_back((hs[i] - mn) / 1e3);
            std::sort(st0.begin(), st0.end());
            fprintf(stderr, "trace: wide-block warps tasks p0 %u p50 %u p99 %u max %u | start us p50 %.1f max %.1f\n", tt[0], tt[tt.size() / 2],
                    tt[tt.size() * 99 / 100], tt.back(), st0[nw / 2], st0[nw - 1]);
            // slowest warp
            int sl = 0;
            for (int i = 0; i < nw; i++) if (h[2 * i] > h[2 * sl]) sl = i;
            fprintf(stderr, "trace: slowest warp %d (block %d) tasks %u work_end %.1f\n", sl, sl / kWarpsPerBlock, ht[sl], (h[2 * sl] - mn) / 1e3);
        }
        std::vector<double> wk, en;
        for (int i = 0; i < nw; i++) { wk.push_back((h[2 * i] - mn) / 1e3); en.push_back((h[2 * i + 1] - mn) / 1e3); }
        std::sort(wk.begin(), wk.end());
        std::sort(en.begin(), en.end());
        fprintf(stderr, "trace: warps=%d blocks_n=%d work_end us: p0 %.1f p10 %.1f p50 %.1f p90 %.1f p100 %.1f | epi end p50 %.1f p100 %.1f\n",
                nw, a.blocks_n, wk[0], wk[nw / 10], wk[nw / 2], wk[nw * 9 / 10], wk[nw - 1], en[nw / 2], en[nw - 1]);
    }
#endif
    return cudaSuccess;
}

template <int VEC, int G, int NV>
cudaError_t run_cell_j(const SpmmArgs &a, cudaStream_t s) {
    return a.J == Layout<VEC, G, NV>::JT ? run_cell<VEC, G, NV, true>(a, s) : run_cell<VEC, G, NV, false>(a, s);
}

template <int VEC, int G, int NV, bool FULL>
cudaError_t run_csr(const lf_csr &A, const float *B, int64_t ldb, int J, float *C, int64_t ldc, cudaStream_t s) {
    static int caps[64];
    auto fn = csr_spmm_kernel<VEC, G, NV, FULL>;
    int &cap = caps[current_device()];
    if (!cap) cap = resident_blocks(fn);
    int64_t want = (A.n_rows + kWarpsPerBlock - 1) / kWarpsPerBlock;
    int grid = (int)std::max<int64_t>(1, std::min<int64_t>(want, cap));
    fn<<<grid, kWarpsPerBlock * 32, 0, s>>>(A.row_ptr, A.col_ind, A.val, A.n_rows, B, ldb, C, ldc, J);
    return cudaGetLastError();
}

template <int VEC, int G, int NV>
cudaError_t run_csr_j(const lf_csr &A, const float *B, int64_t ldb, int J, float *C, int64_t ldc, cudaStream_t s) {
    return J == Layout<VEC, G, NV>::JT ? run_csr<VEC, G, NV, true>(A, B, ldb, J, C, ldc, s)
                                       : run_csr<VEC, G, NV, false>(A, B, ldb, J, C, ldc, s);
}

// ---- grouped (column-merged) path -----------------------------------------
// Eq. 7 charges a bucket U.J for its B reads (U = distinct columns):
// the cost model assumes every distinct B row is fetched once.  The per-slot
// path above fetches one B row per nonzero instead, so on matrices whose
// consecutive rows share columns (banded / FEM / stencil) it gathers each
// B row several times (27-point stencil: every column is in 3 consecutive
// rows).  The grouped path takes kGR consecutive CELL rows of a bucket (W <=
// 32) per warp, merges their columns in a per-warp shared-memory hash table
// (key = column, value = the kGR row values), gathers each DISTINCT B row
// once and applies it to all kGR row accumulators held in registers.
// Measured B-row gathers drop to the group's union (stencil: 0.50 of nnz at
// kGR = 4).  Rows are written like the per-slot path: plain store when the
// CELL row is the whole C row, red.add otherwise (kRowRun rows pre-zeroed).
constexpr int kGR = kGroupRows;  // CELL rows per group
constexpr int kHT = 256;   // hash slots per warp (>= kGR * 32 distinct columns)
#ifndef LF_GROUP_U
#define LF_GROUP_U 2  // distinct columns in flight per lane group (grouped path; 2 measured 1-4% faster than 4)
#endif
constexpr int kGPad = 4 * LF_GROUP_U;  // entry lists padded to a multiple of G * U (G <= 4)
struct GroupStage {
    int32_t key[kHT];      // column in hash slot, -1 = free
    int32_t idx_of[kHT];   // entry index of the slot's column
    int32_t hslot[kGR * 32];
    const float *caddr[kGR * 32 + kGPad];  // entry k: its B row (resolved once) ...
    float4 cval[kGR * 32 + kGPad];         // ... and its value in each of the kGR rows (0 if absent)
};
#ifndef LF_GROUP_MIN_BLOCKS
#define LF_GROUP_MIN_BLOCKS 4
#endif

__device__ __forceinline__ float *f4c(float4 &v, int r) { return reinterpret_cast<float *>(&v) + r; }

template <int G, int NV, bool FULL, bool MD = false>
__global__ void __launch_bounds__(kWarpsPerBlock * 32, LF_GROUP_MIN_BLOCKS) cell_spmm_grouped_kernel(const SpmmArgs a) {
    using Cx = Ctx<4, G, NV, FULL, MD>;
    using V = typename Cx::V;
    using VT = typename Cx::VT;
    using L = Layout<4, G, NV>;
    constexpr int U = LF_GROUP_U;
    static_assert(G * U <= kGPad, "entry padding");
    __shared__ __align__(16) GroupStage gs_all[kWarpsPerBlock];
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    GroupStage &gs = gs_all[w];
    for (int q = lane; q < kHT; q += 32) gs.key[q] = -1;
    __syncwarp();
    const uint64_t pol = policy_evict_first();
    const Cx cx{a.B, a.ldb, a.C, a.ldc, a.J, 0, lane / L::LPR, lane % L::LPR, pol};
    const int64_t nw = (int64_t)gridDim.x * kWarpsPerBlock;
    zero_rows_warp(a.row_mode, a.n_rows, a.C, a.ldc, a.J, true, 1u << kRowEmpty,
                   (int64_t)blockIdx.x * kWarpsPerBlock + w, nw, lane, pol, MD ? a.n_dst : 0, a.dst, a.row_base);
    const unsigned lt = (1u << lane) - 1u;
    const int64_t n = a.n_groups;
    int bcur = 0;
    int sz = claim_size(n, 0, nw, LF_GROUP_CHUNK);
    int64_t g = claim_get(claim_issue(a.ctr + 1, sz, lane));
    int64_t gend = min(g + sz, n);
    while (g < n) {
        while (bcur + 1 < a.nb_g && __ldg(&a.bk_g[bcur + 1].task_off) <= g) bcur++;
        const BucketDev *bk = a.bk_g + bcur;
        const int t = __ldg(&bk->t);
        const int W = 1 << t;
        const int64_t r0 = (g - __ldg(&bk->task_off)) * kGR;  // first CELL row of the group in the bucket
        const int nr = (int)min((int64_t)kGR, __ldg(&bk->n_rows_pad) - r0);
        const int64_t row0 = __ldg(&bk->row_off) + r0;
        const int64_t slot0 = __ldg(&bk->slot_off) + r0 * W;
        const int32_t tag_l = lane < nr ? __ldg(a.row_tag + row0 + lane) : -1;
        // the group's slots: lane j holds slot j of each row (W <= 32)
        int32_t c[kGR];
        float v[kGR];
#pragma unroll
        for (int r = 0; r < kGR; r++) {
            const bool in = r < nr && lane < W;
            c[r] = in ? ld_stream(a.col + slot0 + (int64_t)r * W + lane, pol) : -1;
            v[r] = in ? ld_stream(a.val + slot0 + (int64_t)r * W + lane, pol) : 0.f;
        }
        // merge: every real slot's column is inserted (linear probing); a new
        // column gets the next entry index in (row, lane) order, so entries
        // -- and the gather / summation order -- are deterministic; then each
        // slot adds its value into component r of its column's entry
        int n_u = 0;
#pragma unroll
        for (int r = 0; r < kGR; r++) {
            bool need = c[r] >= 0, ins = false;
            int h = (int)(((uint32_t)c[r] * 0x9E3779B1u) >> 24);
            while (__any_sync(kFull, need)) {
                if (need) {
                    const int prev = atomicCAS(&gs.key[h], -1, c[r]);
                    if (prev == -1) ins = true;
                    if (prev == -1 || prev == c[r]) need = false;
                    else h = (h + 1) & (kHT - 1);
                }
            }
            const unsigned im = __ballot_sync(kFull, ins);
            if (ins) {
                const int k = n_u + __popc(im & lt);
                gs.idx_of[h] = k;
                gs.hslot[k] = h;
                gs.caddr[k] = cx.rowaddr(c[r]);
                gs.cval[k] = make_float4(0.f, 0.f, 0.f, 0.f);
            }
            n_u += __popc(im);
            __syncwarp();
            if (c[r] >= 0) atomicAdd(f4c(gs.cval[gs.idx_of[h]], r), v[r]);
        }
        // pad the entry list to a multiple of G * U with zero entries (the
        // zero row, values 0): the gather loop needs no bounds checks
        const int n_pad = (n_u + G * U - 1) / (G * U) * (G * U);
        if (lane < n_pad - n_u) {
            gs.caddr[n_u + lane] = cx.rowaddr(-1);
            gs.cval[n_u + lane] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
        __syncwarp();
        // gather each distinct B row once; lane group gi takes entries gi, gi + G, ...
        VT acc[kGR][NV];
#pragma unroll
        for (int r = 0; r < kGR; r++) cx.zero(acc[r]);
        for (int k0 = cx.g; k0 < n_pad; k0 += G * U) {
            VT b[U][NV];
            float4 vv[U];
#pragma unroll
            for (int u = 0; u < U; u++) {
                vv[u] = gs.cval[k0 + u * G];
                cx.gather(gs.caddr[k0 + u * G], b[u]);
            }
#pragma unroll
            for (int u = 0; u < U; u++)
#pragma unroll
                for (int m = 0; m < NV; m++) {
                    V::fma(acc[0][m], vv[u].x, b[u][m]);
                    V::fma(acc[1][m], vv[u].y, b[u][m]);
                    V::fma(acc[2][m], vv[u].z, b[u][m]);
                    V::fma(acc[3][m], vv[u].w, b[u][m]);
                }
        }
        for (int k = lane; k < n_u; k += 32) gs.key[gs.hslot[k]] = -1;  // free the used slots
#pragma unroll
        for (int r = 0; r < kGR; r++) {
            cx.reduce_groups(acc[r]);
            const int32_t tag = __shfl_sync(kFull, tag_l, r);
            if (r < nr && tag >= 0 && cx.g == 0) cx.write(a, tag_row(tag), tag_whole(tag), acc[r]);
        }
        __syncwarp();
        if (++g >= gend) {
            sz = claim_size(n, g, nw, LF_GROUP_CHUNK);
            g = claim_get(claim_issue(a.ctr + 1, sz, lane));
            gend = min(g + sz, n);
        }
    }
    if (lane == 0) {  // the last warp out resets the queue counters (as cell_spmm_kernel)
        __threadfence();
        if (atomicAdd(a.ctr + 2, 1ull) == (unsigned long long)gridDim.x * kWarpsPerBlock - 1) {
            __threadfence();
            a.ctr[0] = 0;
            a.ctr[1] = 0;
            a.ctr[2] = 0;
        }
    }
}

template <int G, int NV, bool FULL, bool MD = false>
cudaError_t run_grouped(const SpmmArgs &a, cudaStream_t s) {
    static int caps[64];
    auto fn = cell_spmm_grouped_kernel<G, NV, FULL, MD>;
    int &cap = caps[current_device()];
    if (!cap) cap = resident_blocks(fn);
    const int64_t want = std::max<int64_t>((a.n_groups + kWarpsPerBlock - 1) / kWarpsPerBlock,
                                           (a.n_rows + 32 * kWarpsPerBlock - 1) / (32 * kWarpsPerBlock));
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(cap, want));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(kWarpsPerBlock * 32);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, fn, a);
}

template <int G, int NV>
cudaError_t run_grouped_j(const SpmmArgs &a, cudaStream_t s) {
    return a.J == Layout<4, G, NV>::JT ? run_grouped<G, NV, true>(a, s) : run_grouped<G, NV, false>(a, s);
}

// ---- tensor-core grouped path (mma.sync m16n8k8 TF32, 3xTF32 split) -------
// A group of kMR = 16 consecutive CELL rows of a bucket (W <= 32) is one dense
// contraction: C_group[16 x J] = V[16 x K] . Bg[K x J], K = the group's
// distinct columns (entries) and Bg their B rows.  On banded / dense-block
// matrices K is small (band half-width 12: K = 40 for 16 rows of 25), so
// every B row is gathered about K / 16 = 2.5 times per row of A instead of 25.
// The warp merges the rows' columns in a shared-memory hash set (as the
// grouped path) and scatters the values into V (smem, zero where a row lacks
// the column), then runs the contraction on the tensor cores with fp32
// accuracy from three TF32 products (a_hi b_hi + a_hi b_lo + a_lo b_hi, each
// operand x = hi + lo with hi = tf32(x)); integer-valued inputs are exact.
// Fragment mapping: n-tile j, fragment column n of lane group g = lane / 4
// is C column g * NT + j for B and (2t or 2t+1) * NT + j for D (t = lane % 4),
// so each lane loads NT contiguous floats of a B row (NT / 4 LDG.128) and
// owns 2 NT contiguous floats of its two C rows (g, g + 8).  A group whose K
// exceeds kKCap is computed by the plain per-slot loop instead.
constexpr int kMR = 16;           // rows per tensor-core group (MMA M)
constexpr int kKCap = 64;         // max distinct columns per group
constexpr int kMHT = 128;         // hash slots (<= kKCap + 32 keys ever inserted)
constexpr int kVStride = kKCap + 4;  // V row stride (floats): conflict-free A-fragment loads
constexpr int kMmaWarps = 4;
struct MmaStage {
    int32_t key[kMHT];
    int32_t idx_of[kMHT];
    int32_t hslot[kKCap + 32];
    const float *caddr[kKCap + 32];  // entries up to kKCap + 31 are written before `over` is seen
    float V[kMR * kVStride];
};

__device__ __forceinline__ uint32_t tf32_hi(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return r;
}
__device__ __forceinline__ void split_tf32(float x, uint32_t &hi, uint32_t &lo) {
    hi = tf32_hi(x);
    lo = tf32_hi(x - __uint_as_float(hi));
}
__device__ __forceinline__ void mma_tf32(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
    asm volatile(
        "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
        "{%0,%1,%2,%3};"
        : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

template <int NT>
__global__ void __launch_bounds__(kMmaWarps * 32) cell_spmm_mma_kernel(const SpmmArgs a) {
    const int J = a.J;  // a multiple of 8 NT
    __shared__ __align__(16) MmaStage ms_all[kMmaWarps];
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    MmaStage &ms = ms_all[w];
    for (int q = lane; q < kMHT; q += 32) ms.key[q] = -1;
    __syncwarp();
    const uint64_t pol = policy_evict_first();
    const int64_t nw = (int64_t)gridDim.x * kMmaWarps;
    zero_rows_warp(a.row_mode, a.n_rows, a.C, a.ldc, a.J, true, 1u << kRowEmpty,
                   (int64_t)blockIdx.x * kMmaWarps + w, nw, lane, pol);
    const unsigned lt = (1u << lane) - 1u;
    const int g = lane >> 2, t = lane & 3;
    const float *zrow = reinterpret_cast<const float *>(g_zero_row);
    const int64_t n = a.n_groups_m;
    int bcur = 0;
    int sz = claim_size(n, 0, nw);
    int64_t grp = claim_get(claim_issue(a.ctr + 1, sz, lane));
    int64_t gend = min(grp + sz, n);
    while (grp < n) {
        while (bcur + 1 < a.nb_g && __ldg(&a.bk_m[bcur + 1].task_off) <= grp) bcur++;
        const BucketDev *bk = a.bk_m + bcur;
        const int W = 1 << __ldg(&bk->t);
        const int64_t r0 = (grp - __ldg(&bk->task_off)) * kMR;
        const int nr = (int)min((int64_t)kMR, __ldg(&bk->n_rows_pad) - r0);
        const int64_t row0 = __ldg(&bk->row_off) + r0;
        const int64_t slot0 = __ldg(&bk->slot_off) + r0 * W;
        const int32_t tag_l = lane < nr ? __ldg(a.row_tag + row0 + lane) : -1;
        for (int q = lane; q < kMR * kVStride / 4; q += 32)
            reinterpret_cast<float4 *>(ms.V)[q] = make_float4(0.f, 0.f, 0.f, 0.f);
        // merge the rows' columns (rows in order, lanes in order: entries numbered
        // deterministically); V[r][entry] += value
        int n_u = 0;
        bool over = false;
        int32_t cr[kMR];
        float vr[kMR];
#pragma unroll
        for (int r = 0; r < kMR; r++) {  // all the group's slots in flight at once
            const bool in = r < nr && lane < W;
            cr[r] = in ? ld_stream(a.col + slot0 + (int64_t)r * W + lane, pol) : -1;
            vr[r] = in ? ld_stream(a.val + slot0 + (int64_t)r * W + lane, pol) : 0.f;
        }
#pragma unroll
        for (int r = 0; r < kMR; r++) {
            if (over) break;
            const int32_t c = cr[r];
            const float v = vr[r];
            bool need = c >= 0, ins = false;
            int h = (int)(((uint32_t)c * 0x9E3779B1u) >> 25);  // 7 bits: kMHT = 128
            while (__any_sync(kFull, need)) {
                if (need) {
                    const int prev = atomicCAS(&ms.key[h], -1, c);
                    if (prev == -1) ins = true;
                    if (prev == -1 || prev == c) need = false;
                    else h = (h + 1) & (kMHT - 1);
                }
            }
            const unsigned im = __ballot_sync(kFull, ins);
            if (ins) {
                const int k = n_u + __popc(im & lt);
                ms.idx_of[h] = k;
                ms.hslot[k] = h;
                ms.caddr[k] = k < kKCap ? a.B + (int64_t)c * a.ldb : zrow;
            }
            n_u += __popc(im);
            __syncwarp();
            over = n_u > kKCap;
            if (!over && c >= 0) atomicAdd(&ms.V[r * kVStride + ms.idx_of[h]], v);
        }
        __syncwarp();
        if (!over) {
            const int n_pad = (n_u + 7) & ~7;
            if (lane < n_pad - n_u) ms.caddr[n_u + lane] = zrow;
            __syncwarp();
            // J in slices of 8 NT columns; per slice the k-steps run with the
            // next step's B rows loaded before this step's products
            for (int jp = 0; jp < a.J; jp += 8 * NT) {
                float acc[NT][4];
#pragma unroll
                for (int j = 0; j < NT; j++) acc[j][0] = acc[j][1] = acc[j][2] = acc[j][3] = 0.f;
                float b0[NT], b1[NT], n0[NT], n1[NT];
                auto load_b = [&](int k0, float (&x0)[NT], float (&x1)[NT]) {
                    const float *e0 = ms.caddr[k0 + t], *e1 = ms.caddr[k0 + t + 4];
                    const bool z0 = e0 == zrow, z1 = e1 == zrow;
#pragma unroll
                    for (int q = 0; q < NT; q += 4) {
                        const float4 y0 = z0 ? make_float4(0.f, 0.f, 0.f, 0.f)
                                             : __ldg(reinterpret_cast<const float4 *>(e0 + jp + g * NT + q));
                        const float4 y1 = z1 ? make_float4(0.f, 0.f, 0.f, 0.f)
                                             : __ldg(reinterpret_cast<const float4 *>(e1 + jp + g * NT + q));
                        x0[q] = y0.x, x0[q + 1] = y0.y, x0[q + 2] = y0.z, x0[q + 3] = y0.w;
                        x1[q] = y1.x, x1[q + 1] = y1.y, x1[q + 2] = y1.z, x1[q + 3] = y1.w;
                    }
                };
                if (n_pad > 0) load_b(0, n0, n1);
                for (int k0 = 0; k0 < n_pad; k0 += 8) {
#pragma unroll
                    for (int j = 0; j < NT; j++) {
                        b0[j] = n0[j];
                        b1[j] = n1[j];
                    }
                    if (k0 + 8 < n_pad) load_b(k0 + 8, n0, n1);
                    uint32_t ah[4], al[4];
                    split_tf32(ms.V[g * kVStride + k0 + t], ah[0], al[0]);
                    split_tf32(ms.V[(g + 8) * kVStride + k0 + t], ah[1], al[1]);
                    split_tf32(ms.V[g * kVStride + k0 + t + 4], ah[2], al[2]);
                    split_tf32(ms.V[(g + 8) * kVStride + k0 + t + 4], ah[3], al[3]);
#pragma unroll
                    for (int j = 0; j < NT; j++) {
                        uint32_t bh0, bl0, bh1, bl1;
                        split_tf32(b0[j], bh0, bl0);
                        split_tf32(b1[j], bh1, bl1);
                        mma_tf32(acc[j], al, bh0, bh1);
                        mma_tf32(acc[j], ah, bl0, bl1);
                        mma_tf32(acc[j], ah, bh0, bh1);
                    }
                }
                // rows g and g + 8: columns jp + [2t NT, 2t NT + 2 NT)
#pragma unroll
                for (int half = 0; half < 2; half++) {
                    const int r = g + 8 * half;
                    const int32_t tag = __shfl_sync(kFull, tag_l, r);
                    if (r < nr && tag >= 0) {
                        float *p = a.C + (int64_t)tag_row(tag) * a.ldc + jp + 2 * t * NT;
                        const bool plain = tag_whole(tag);
#pragma unroll
                        for (int q = 0; q < NT; q += 4) {
                            const float4 lo4 = make_float4(acc[q][2 * half], acc[q + 1][2 * half],
                                                           acc[q + 2][2 * half], acc[q + 3][2 * half]);
                            const float4 hi4 = make_float4(acc[q][2 * half + 1], acc[q + 1][2 * half + 1],
                                                           acc[q + 2][2 * half + 1], acc[q + 3][2 * half + 1]);
                            if (plain) {
                                Vec<4>::store(p + q, lo4, pol);
                                Vec<4>::store(p + NT + q, hi4, pol);
                            } else {
                                Vec<4>::red(p + q, lo4);
                                Vec<4>::red(p + NT + q, hi4);
                            }
                        }
                    }
                }
            }
        } else {
            // too many distinct columns: the rows one by one, per slot (lane
            // covers 4 of the J columns; J = 8 NT <= 128)
            for (int r = 0; r < nr; r++) {
                const int32_t tag = __shfl_sync(kFull, tag_l, r);
                if (tag < 0) continue;
                const int32_t c = lane < W ? ld_stream(a.col + slot0 + (int64_t)r * W + lane, pol) : -1;
                const float v = lane < W ? ld_stream(a.val + slot0 + (int64_t)r * W + lane, pol) : 0.f;
                float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
                for (int q = 0; q < W; q++) {
                    const int32_t cq = __shfl_sync(kFull, c, q);
                    const float vq = __shfl_sync(kFull, v, q);
                    if (cq < 0 || 4 * lane >= J) continue;
                    Vec<4>::fma(s, vq, __ldg(reinterpret_cast<const float4 *>(a.B + (int64_t)cq * a.ldb) + lane));
                }
                if (4 * lane < J) {
                    float *p = a.C + (int64_t)tag_row(tag) * a.ldc + 4 * lane;
                    if (tag_whole(tag)) Vec<4>::store(p, s, pol);
                    else Vec<4>::red(p, s);
                }
            }
        }
        for (int k = lane; k < n_u; k += 32) ms.key[ms.hslot[k]] = -1;  // free the used slots
        __syncwarp();
        if (++grp >= gend) {
            sz = claim_size(n, grp, nw);
            grp = claim_get(claim_issue(a.ctr + 1, sz, lane));
            gend = min(grp + sz, n);
        }
    }
    if (lane == 0) {  // the last warp out resets the queue counters (as cell_spmm_kernel)
        __threadfence();
        if (atomicAdd(a.ctr + 2, 1ull) == (unsigned long long)gridDim.x * kMmaWarps - 1) {
            __threadfence();
            a.ctr[0] = 0;
            a.ctr[1] = 0;
            a.ctr[2] = 0;
        }
    }
}

template <int NT>
cudaError_t run_mma(const SpmmArgs &a, cudaStream_t s) {
    static int caps[64];
    auto fn = cell_spmm_mma_kernel<NT>;
    int &cap = caps[current_device()];
    if (!cap) {
        int occ = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, kMmaWarps * 32, 0);
        cap = std::max(1, occ) * sm_count();
    }
    const int64_t want = std::max<int64_t>((a.n_groups_m + kMmaWarps - 1) / kMmaWarps,
                                           (a.n_rows + 32 * kMmaWarps - 1) / (32 * kMmaWarps));
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(cap, want));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(kMmaWarps * 32);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, fn, a);
}

// c_bits: OR of every C base address the launch writes (C, or each fused-exchange destination)
bool vec8_ok(const float *B, int64_t ldb, uintptr_t c_bits, int64_t ldc, int J) {
    return J % 8 == 0 && ldb % 8 == 0 && ldc % 8 == 0 && ((uintptr_t)B & 31) == 0 && (c_bits & 31) == 0;
}

bool vec4_ok(const float *B, int64_t ldb, uintptr_t c_bits, int64_t ldc, int J) {
    return J % 4 == 0 && ldb % 4 == 0 && ldc % 4 == 0 && ((uintptr_t)B & 15) == 0 && (c_bits & 15) == 0;
}

bool vec4_ok(const float *B, int64_t ldb, const float *C, int64_t ldc, int J) {
    return vec4_ok(B, ldb, (uintptr_t)C, ldc, J);
}

}  // namespace
}  // namespace lf

namespace lf {
// cross-TU entry points (cell_spmm*.cu)
cudaError_t zero_red_rows(const SpmmArgs &a, bool tiled, cudaStream_t s);
bool grouped_ok(const SpmmArgs &a);
bool mma_ok(const SpmmArgs &a);
cudaError_t spmm_v8(const SpmmArgs &a, cudaStream_t s);        // cell_spmm_v8.cu
cudaError_t spmm_grouped(const SpmmArgs &a, cudaStream_t s);   // cell_spmm_grp.cu
cudaError_t spmm_mma(const SpmmArgs &a, cudaStream_t s);       // cell_spmm_grp.cu
cudaError_t spmm_md(const SpmmArgs &a, bool v4, cudaStream_t s);  // cell_spmm_md.cu
}  // namespace lf
