// cell_spmm_tc.cu -- the CELL SpMM of "windowed" row groups on the 5th-
// generation tensor cores (tcgen05, kind::tf32, fp32-accurate 3xTF32 split),
// SURVEY 8(a) rows a6/a7, 8(f) NEXT-4; DESIGN.md section 7 "Tensor-core path".
//
// A group is kTcN = 128 consecutive CELL rows of one bucket (W <= 32).  Its
// real column indices lie in a WINDOW [lo, lo + span) of B rows (per-group
// table built by tc_window_kernel at lf_cell_build).  On banded / FEM-like
// matrices the window is short (half-width-12 band: span = 152 for 128 rows),
// so the group is one dense contraction over the window (eq. 4):
//
//     C[rows]^T  (J x 128)  =  Bwin^T (J x span)  .  V^T (span x 128)
//
// with V[n][k] = value of CELL row n at column lo + k (0 where absent) and
// Bwin the window's B rows.  Every B row of the window is read ONCE per group
// (the U.J term of eq. 7, rather than one gather per nonzero).
// Mapping (all measured conventions checked by tools/tc_probe.cu on B200):
//   * A operand = Bwin^T in TMEM: lane j (= output column), column k.  Loader
//     warps read 32 window rows of B (coalesced: lane j reads B[k][j]), split
//     x = hi + lo (the tensor core TRUNCATES fp32 to tf32, so hi = x itself and
//     lo = x - trunc_tf32(x)) and store both with tcgen05.st (STTM);
//   * B operand = V^T in shared memory, K-major, 128-byte swizzle: builder
//     threads (one per CELL row) write their row's dense 32-column chunk (raw
//     value and lo part);
//   * D = C^T in TMEM (lane j, column n), double buffered; one thread issues
//     D += A_hi.V_hi + A_lo.V_hi + A_hi.V_lo per 8-deep k step (UTCHMMA); the
//     missing lo.lo term is 2^-20 relative (3xTF32), well inside 1e-5;
//   * epilogue warps read D with tcgen05.ld (LDTM): thread j holds column j
//     of 32 rows, so each C row slice is a coalesced 128-byte warp store
//     (red.global.add for rows several CELL rows sum into, as the grouped path).
// Warp roles (one 416-thread CTA per SM, persistent, static round-robin over
// groups): 0-3 loaders (TMEM lanes 32w..), 4-7 epilogue (lanes 32(w%4)..),
// 8-11 V builders, 12 MMA issuer + TMEM allocator.  Pipelines: a 4-stage ring
// of (A chunk in TMEM, V chunk in smem) and 2 accumulators, each with
// full/empty mbarriers (tcgen05.commit arrives on the empty ones).
// A group whose window exceeds kTcMaxChunks * 32 rows is computed by the
// builder warps on the CUDA cores instead (same result up to fp32 order).
#include "../lf_internal.cuh"

#include <cstdio>
#include <vector>

namespace lf {

namespace {

constexpr int kTcN = 128;       // CELL rows per group (MMA N)
constexpr int kTcK = 32;        // window rows per pipeline stage
constexpr int kTcAStages = 4;   // A chunks (B window rows, raw + lo) in TMEM
constexpr int kTcVStages = 3;   // V^T chunks in smem
constexpr int kTcBStages = 4;   // B window chunks landed by TMA in smem
constexpr int kTcCStages = 2;   // a group's CELL rows (cols, vals) landed by TMA in smem
constexpr int kTcMaxChunks = 8; // window cap: 256 B rows per group
constexpr int kTcMaxJ = 128;
constexpr int kNBuild = 8;                // V builder warps
constexpr int kBRows = kTcN / kNBuild;    // CELL rows per builder warp
constexpr int kTcWarps = 8 + kNBuild + 2;
constexpr int kWEpi = 4, kWBuild = 8, kWMma = kWBuild + kNBuild, kWTma = kWMma + 1;
constexpr uint32_t kTmemCols = 512;  // D: 2 x 128, A: kTcAStages x 64 (raw 32 + lo 32)
constexpr uint32_t kColA = 256;
constexpr unsigned kFull = 0xffffffffu;
constexpr int kCellWords = kTcN * 32 + 8;  // a group's slots (W <= 32) + alignment slack of the bulk copy

struct TcShared {
    float vhi[kTcVStages][kTcN * kTcK];  // V^T chunk, raw values (K-major SW128), 16 KB each
    float vlo[kTcVStages][kTcN * kTcK];  // V^T chunk, lo parts
    float bwin[kTcBStages][kTcK * kTcMaxJ];  // B window chunk: 32 rows x J, row-major (packed)
    int32_t ccol[kTcCStages][kCellWords];    // group's colInd slots
    float cval[kTcCStages][kCellWords];      // group's val slots
    unsigned long long full_a[kTcAStages], empty_a[kTcAStages];
    unsigned long long full_v[kTcVStages], empty_v[kTcVStages];
    unsigned long long full_b[kTcBStages], empty_b[kTcBStages];
    unsigned long long full_c[kTcCStages], empty_c[kTcCStages];
    unsigned long long full_d[2], empty_d[2];
    // which window rows a group references (byte k: B row lo + k), written by
    // the builders, double buffered by group parity: the loaders pass only those rows
    // and put exact zeros elsewhere, so a B row no nonzero references never
    // enters the contraction (0 x NaN would) -- Alg. 1 never reads it either
    uint8_t ref[2][kTcMaxChunks * kTcK];  // 1 = window row referenced
    unsigned long long full_m[2], empty_m[2];
    uint32_t tmem;
};
constexpr size_t kTcSmem = sizeof(TcShared);
static_assert(kTcSmem <= 232448, "shared memory of one CTA");

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

// ---- mbarrier ----
__device__ __forceinline__ void mbar_init(unsigned long long *b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long *b) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
// the retry loop is C++ (not a branch inside the asm), so the compiler sees a
// structured loop and knows the warp reconverges after it -- warp-synchronous
// intrinsics that follow are then not lowered to the slow divergent fallback
// a waiting warp sleeps in hardware until the phase completes (or this
// hint elapses) instead of re-issuing try_wait: spinning waiters would take
// issue slots from the builder and epilogue warps
constexpr uint32_t kSuspendNs = 1000000;
__device__ __forceinline__ bool mbar_try_wait(unsigned long long *b, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n.reg .pred p;\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n"
        "selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(smem_u32(b)), "r"(parity), "r"(kSuspendNs)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(unsigned long long *b, uint32_t parity) {
    while (!mbar_try_wait(b, parity)) {
    }
}
#ifdef LF_TC_TRACE
// diagnostic builds: cycles each role spends waiting on each barrier, per CTA
__device__ unsigned long long lf_tc_trace[1024][24];
#define TC_WAIT(slot, bar, par)                                               \
    do {                                                                      \
        const long long t0_ = clock64();                                      \
        mbar_wait(bar, par);                                                  \
        if ((threadIdx.x & 31) == 0) atomicAdd(&lf_tc_trace[blockIdx.x][slot], (unsigned long long)(clock64() - t0_)); \
    } while (0)
#else
#define TC_WAIT(slot, bar, par) mbar_wait(bar, par)
#endif
__device__ __forceinline__ void mbar_expect_tx(unsigned long long *b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
// TMA 1-D bulk copy global -> shared, completing `bytes` on the mbarrier
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, unsigned long long *b) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(b))
        : "memory");
}

// ---- tcgen05 ----
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(unsigned long long *b) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(b))
                 : "memory");
}
// D[tmem] (+)= A[tmem] . B[smem desc]   (kind::tf32, M = 128, N = kTcN)
__device__ __forceinline__ void tc_mma(uint32_t d, uint32_t a, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\n"
        "tcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}" ::"r"(d),
        "r"(a), "l"(bdesc), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void tmem_st32(uint32_t t, const uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
        "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(t),
        "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]),
        "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]),
        "r"(r[18]), "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]),
        "r"(r[26]), "r"(r[27]), "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
        : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t t, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,"
        "%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(t));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// K-major, 128-byte swizzle smem descriptor (tile base 1024-aligned): start
// address, LBO 16 B (unused for swizzled K-major), SBO 1024 B (8 rows x 128 B),
// version 1 (sm_100), layout SWIZZLE_128B
__device__ __forceinline__ uint64_t sw128_desc(const void *tile) {
    const uint64_t a = smem_u32(tile);
    return ((a >> 4) & 0x3FFF) | (1ull << 16) | (64ull << 32) | (1ull << 46) | (2ull << 61);
}
__device__ __forceinline__ float tf32_lo(float x) { return x - __uint_as_float(__float_as_uint(x) & 0xffffe000u); }

__device__ __forceinline__ void grid_dep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void st_f32(float *p, float v, uint64_t pol) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(p), "f"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ void red_f32(float *p, float v) {
    asm volatile("red.global.add.f32 [%0], %1;" ::"l"(p), "f"(v) : "memory");
}

// group g: bucket (cursor moves forward: every role walks g increasing)
struct TcGroup {
    int64_t row0, slot0;
    int t, nr, lo, span, nch;
    bool mma;  // contracted on the tensor cores (else: empty, or the CUDA-core fallback)
};
__device__ __forceinline__ TcGroup tc_group(const SpmmArgs &a, int64_t g, int &bcur) {
    while (bcur + 1 < a.nb_t && __ldg(&a.bk_t[bcur + 1].task_off) <= g) bcur++;
    const BucketDev *bk = a.bk_t + bcur;
    TcGroup x;
    x.t = __ldg(&bk->t);
    const int64_t r0 = (g - __ldg(&bk->task_off)) * kTcN;
    x.nr = (int)min((int64_t)kTcN, __ldg(&bk->n_rows_pad) - r0);
    x.row0 = __ldg(&bk->row_off) + r0;
    x.slot0 = __ldg(&bk->slot_off) + (r0 << x.t);
    const int2 w = __ldg(a.tc_win + g);  // {lo, span}; span 0: no real slot
    x.lo = w.x;
    x.span = w.y;
    x.nch = (x.span + kTcK - 1) / kTcK;
    x.mma = x.span > 0 && x.nch <= kTcMaxChunks;
    return x;
}

// The CTA's groups g = blockIdx.x, + gridDim.x, ...; the NEXT group's
// descriptor is fetched when a group starts, so its global loads (bucket
// table, window) are in flight while the current group is processed instead
// of stalling every role at every group boundary.
struct TcIter {
    int64_t g, n;
    int bcur;
    TcGroup x, nx;
    __device__ __forceinline__ TcIter(const SpmmArgs &a) : g(blockIdx.x), n(a.n_groups_t), bcur(0) {
        if (g < n) x = tc_group(a, g, bcur);
        if (g + gridDim.x < n) nx = tc_group(a, g + gridDim.x, bcur);
    }
    __device__ __forceinline__ void next(const SpmmArgs &a) {
        g += gridDim.x;
        x = nx;
        if (g + gridDim.x < n) nx = tc_group(a, g + gridDim.x, bcur);
    }
};

__device__ __forceinline__ bool tag_whole(int32_t tag) { return (tag & 7) == 7; }
__device__ __forceinline__ int32_t tag_row(int32_t tag) { return tag >> 3; }

// rows of A with no CELL row are +0.0 (R13): the builder warps zero their share
__device__ void zero_empty_rows(const SpmmArgs &a, int64_t wid, int64_t nw, int lane, uint64_t pol) {
    for (int64_t base = wid * 32; base < a.n_rows; base += nw * 32) {
        const int64_t i = base + lane;
        unsigned need = __ballot_sync(kFull, i < a.n_rows && __ldg(a.row_mode + i) == kRowEmpty);
        while (need) {
            const int src = __ffs(need) - 1;
            need &= need - 1;
            for (int d = 0; d < max(a.n_dst, 1); d++) {  // C, or every fused-exchange destination
                float *row = (a.n_dst ? ld_dst(a.dst, d) + a.row_base * a.ldc : a.C) + (base + src) * a.ldc;
                for (int j = lane * 4; j < a.J; j += 128)
                    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.f32 [%0], {%1, %1, %1, %1}, %2;" ::"l"(
                                     row + j),
                                 "f"(0.f), "l"(pol)
                                 : "memory");
            }
        }
    }
}

// CUDA-core fallback for a group whose window is too wide: builder warp w
// takes rows w, w + kNBuild, ...; lanes split J into float4 (J <= 128, J % 4 == 0)
__device__ void fallback_group(const SpmmArgs &a, const TcGroup &x, int bw, int lane, uint64_t pol) {
    const int W = 1 << x.t;
    const int j = 4 * lane;
    for (int n = bw; n < x.nr; n += kNBuild) {
        const int32_t tag = __ldg(a.row_tag + x.row0 + n);
        if (tag < 0) continue;
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        for (int w = 0; w < W; w++) {
            const int32_t c = __ldg(a.col + x.slot0 + (int64_t)n * W + w);
            if (c < 0) break;  // padding slots are a suffix
            const float v = __ldg(a.val + x.slot0 + (int64_t)n * W + w);
            if (j < a.J) {
                const float4 b = __ldg(reinterpret_cast<const float4 *>(a.B + (int64_t)c * a.ldb + j));
                acc.x = fmaf(v, b.x, acc.x);
                acc.y = fmaf(v, b.y, acc.y);
                acc.z = fmaf(v, b.z, acc.z);
                acc.w = fmaf(v, b.w, acc.w);
            }
        }
        for (int d = 0; d < max(a.n_dst, 1) && j < a.J; d++) {
            float *p = (a.n_dst ? ld_dst(a.dst, d) + a.row_base * a.ldc : a.C) + (int64_t)tag_row(tag) * a.ldc + j;
            if (tag_whole(tag)) {
                asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p),
                             "f"(acc.x), "f"(acc.y), "f"(acc.z), "f"(acc.w), "l"(pol)
                             : "memory");
            } else {
                grid_dep_wait();
                asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(acc.x), "f"(acc.y),
                             "f"(acc.z), "f"(acc.w)
                             : "memory");
            }
        }
    }
}

__global__ void __launch_bounds__(kTcWarps * 32, 1) cell_spmm_tc_kernel(const SpmmArgs a) {
    // dynamic shared memory starts at the CTA's (1024-aligned) shared window
    // base: no static __shared__ in this kernel.  Addressing it through the
    // __shared__ symbol (no integer round trip) keeps every access an LDS/STS
    // instead of a generic LD/ST.
    extern __shared__ __align__(1024) uint8_t smem_raw[];
    TcShared &sm = *reinterpret_cast<TcShared *>(smem_raw);
    if (smem_u32(smem_raw) & 1023) __trap();  // the SW128 tiles need a 1024-byte aligned base
    // warp index broadcast from lane 0: provably warp-uniform, so the role
    // branches below do not make the compiler treat the warps as divergent
    const int warp = __shfl_sync(kFull, (int)(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
#ifdef LF_TC_TRACE
    const long long t_start = clock64();
#endif
    if (warp == kWMma) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&sm.tmem)),
                     "r"(kTmemCols)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    if (threadIdx.x == 0) {
        for (int s = 0; s < kTcAStages; s++) {
            mbar_init(&sm.full_a[s], 4);
            mbar_init(&sm.empty_a[s], 1);
        }
        for (int s = 0; s < kTcVStages; s++) {
            mbar_init(&sm.full_v[s], kNBuild);
            mbar_init(&sm.empty_v[s], 1);
        }
        for (int s = 0; s < kTcBStages; s++) {
            mbar_init(&sm.full_b[s], 1);
            mbar_init(&sm.empty_b[s], 4);
        }
        for (int s = 0; s < kTcCStages; s++) {
            mbar_init(&sm.full_c[s], 1);
            mbar_init(&sm.empty_c[s], kNBuild);
        }
        for (int d = 0; d < 2; d++) {
            mbar_init(&sm.full_d[d], 1);
            mbar_init(&sm.empty_d[d], 4);
            mbar_init(&sm.full_m[d], kNBuild);
            mbar_init(&sm.empty_m[d], 4);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = sm.tmem;
    const int64_t n_groups = a.n_groups_t;
    const uint64_t pol = policy_evict_first();

    if (warp < kWEpi) {
        // ===== loaders: landed B window chunk (smem) -> TMEM A operand, raw + lo =====
        const int j = 32 * warp + lane;
        const bool jok = j < a.J;
        const uint32_t lane_base = tmem + ((uint32_t)(32 * warp) << 16);
        uint32_t sa = 0, pha = 0, sb = 0, phb = 0, mb = 0, phm = 0;
        for (TcIter it(a); it.g < n_groups; it.next(a)) {
            const TcGroup &x = it.x;
            if (!x.mma) continue;
            TC_WAIT(0, &sm.full_m[mb], phm);
            for (int c = 0; c < x.nch; c++) {
                uint32_t fw[8];  // the chunk's 32 reference flags, 4 per word
#pragma unroll
                for (int q = 0; q < 8; q++) fw[q] = jok ? reinterpret_cast<const uint32_t *>(sm.ref[mb] + kTcK * c)[q] : 0u;
                TC_WAIT(1, &sm.full_b[sb], phb);
                const float *tile = sm.bwin[sb] + j;
                uint32_t raw[32], lo[32];
#pragma unroll
                for (int kk = 0; kk < 32; kk++)  // lane j reads word kk * J + j: conflict-free
                    raw[kk] = ((fw[kk >> 2] >> (8 * (kk & 3))) & 0xffu) ? __float_as_uint(tile[kk * a.J]) : 0u;
                __syncwarp();
                if (lane == 0) mbar_arrive(&sm.empty_b[sb]);
                if (++sb == kTcBStages) {
                    sb = 0;
                    phb ^= 1;
                }
#pragma unroll
                for (int kk = 0; kk < 32; kk++) lo[kk] = __float_as_uint(tf32_lo(__uint_as_float(raw[kk])));
                TC_WAIT(2, &sm.empty_a[sa], pha ^ 1);
                tc_fence_after();
                tmem_st32(lane_base + kColA + 64 * sa, raw);
                tmem_st32(lane_base + kColA + 64 * sa + 32, lo);
                asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
                tc_fence_before();
                __syncwarp();
                if (lane == 0) mbar_arrive(&sm.full_a[sa]);
                if (++sa == kTcAStages) {
                    sa = 0;
                    pha ^= 1;
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&sm.empty_m[mb]);
            mb ^= 1;
            if (mb == 0) phm ^= 1;
        }
    } else if (warp < kWBuild) {
        // ===== epilogue: D (TMEM) -> C rows =====
        const int q = warp & 3;
        const int j = 32 * q + lane;
        const bool jok = j < a.J;
        const uint32_t lane_base = tmem + ((uint32_t)(32 * q) << 16);
        uint32_t d = 0, phd = 0;
        for (TcIter it(a); it.g < n_groups; it.next(a)) {
            const TcGroup &x = it.x;
            if (!x.mma) continue;
            int32_t tags[kTcN / 32];
#pragma unroll
            for (int nb = 0; nb < kTcN / 32; nb++)
                tags[nb] = 32 * nb + lane < x.nr ? __ldg(a.row_tag + x.row0 + 32 * nb + lane) : -1;
            TC_WAIT(3, &sm.full_d[d], phd);
            tc_fence_after();
#pragma unroll
            for (int nb = 0; nb < kTcN / 32; nb++) {
                if (32 * nb >= x.nr) break;
                uint32_t v[32];
                tmem_ld32(lane_base + 128 * d + 32 * nb, v);
                if (nb == kTcN / 32 - 1 || 32 * (nb + 1) >= x.nr) {  // accumulator drained: release it
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&sm.empty_d[d]);
                }
                // 32 rows: lane i formed row i's C offset before the wait; each
                // row's offset is shuffled and stored with no compiler barrier in
                // between (plain intrinsics, no asm "memory" clobbers), so the
                // rows pipeline.  Rows several CELL rows add into (pre-zeroed,
                // red.add) are rare: one vote per 32 rows picks the plain loop.
                const int32_t tg = tags[nb];
                const bool whole = tg < 0 || tag_whole(tg);
                const long long roff = tg >= 0 ? (long long)tag_row(tg) * a.ldc : -1;
                // C, or (fused row exchange) each destination C in turn
                for (int dd = 0; dd < max(a.n_dst, 1); dd++) {
                    float *const cb = (a.n_dst ? ld_dst(a.dst, dd) + a.row_base * a.ldc : a.C) + j;
                    if (__all_sync(kFull, whole)) {
#pragma unroll
                        for (int i = 0; i < 32; i++) {
                            const long long ro = __shfl_sync(kFull, roff, i);
                            if (ro >= 0 && jok) __stcs(cb + ro, __uint_as_float(v[i]));
                        }
                    } else {
                        grid_dep_wait();
#pragma unroll
                        for (int i = 0; i < 32; i++) {
                            const long long ro = __shfl_sync(kFull, roff, i);
                            const bool wh = __shfl_sync(kFull, whole, i);
                            if (ro >= 0 && jok) {
                                if (wh) __stcs(cb + ro, __uint_as_float(v[i]));
                                else atomicAdd(cb + ro, __uint_as_float(v[i]));
                            }
                        }
                    }
                }
            }
            d ^= 1;
            if (d == 0) phd ^= 1;
        }
    } else if (warp < kWMma) {
        // ===== V builders: warp bw owns CELL rows kBRows bw .. + kBRows - 1 of a
        // group; lane w = slot w of a row (the landed CELL rows are read
        // conflict-free); the scatter is branch-free so rows interleave (ILP) =====
        const int bw = warp - kWBuild;
        zero_empty_rows(a, (int64_t)blockIdx.x * kNBuild + bw, (int64_t)gridDim.x * kNBuild, lane, pol);
        uint32_t sv = 0, phv = 0, mb = 0, phm = 0, sc = 0, phc = 0;
        for (TcIter it(a); it.g < n_groups; it.next(a)) {
#ifdef LF_TC_TRACE
            long long tb0 = clock64();
#endif
            const TcGroup &x = it.x;
            if (x.span == 0) continue;
            if (!x.mma) {
                fallback_group(a, x, bw, lane, pol);
                continue;
            }
            const int W = 1 << x.t;
            const int off = (int)(x.slot0 & 3);  // the bulk copy starts at a 16-byte boundary
            TC_WAIT(4, &sm.full_c[sc], phc);
#ifdef LF_TC_TRACE
            tb0 = clock64();
#endif
            // rows kBRows bw + r: column (window-relative, -1 = none) and value of slot `lane`
            int32_t col[kBRows];
            float val[kBRows];
            bool dup = false;
#pragma unroll
            for (int r = 0; r < kBRows; r++) {
                const int n = kBRows * bw + r;
                const bool in = n < x.nr && lane < W;
                const int base = off + n * W + lane;
                const int32_t cg = in ? sm.ccol[sc][base] : -1;
                const int32_t cp = in && lane > 0 ? sm.ccol[sc][base - 1] : -1;
                col[r] = cg >= 0 ? cg - x.lo : -1;
                val[r] = in ? sm.cval[sc][base] : 0.f;
                dup = dup || (cg >= 0 && cp == cg);
            }
            if (__any_sync(kFull, dup)) {
                // duplicate columns (kept and summed) are adjacent slots: fold each
                // run into its last slot (segmented inclusive sum; rare)
#pragma unroll
                for (int r = 0; r < kBRows; r++) {
#pragma unroll
                    for (int o = 1; o < 32; o <<= 1) {
                        const float vu = __shfl_up_sync(kFull, val[r], o);
                        const int32_t cu = __shfl_up_sync(kFull, col[r], o);
                        if (lane >= o && cu == col[r] && col[r] >= 0) val[r] += vu;
                    }
                    const int32_t cn = __shfl_down_sync(kFull, col[r], 1);
                    if (lane < 31 && cn == col[r]) col[r] = -1;  // not the last of its run
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&sm.empty_c[sc]);
            if (++sc == kTcCStages) {
                sc = 0;
                phc ^= 1;
            }
            // referenced window rows -> byte flags (idempotent plain stores, no
            // read-modify-write): the builder warps clear the buffer, meet on a
            // named barrier, then flag their rows' columns
            TC_WAIT(5, &sm.empty_m[mb], phm ^ 1);
            if (lane < kTcMaxChunks * kTcK / 4 / kNBuild)
                reinterpret_cast<uint32_t *>(sm.ref[mb])[(kTcMaxChunks * kTcK / 4 / kNBuild) * bw + lane] = 0u;
            asm volatile("bar.sync 1, %0;" ::"n"(kNBuild * 32) : "memory");
#pragma unroll
            for (int r = 0; r < kBRows; r++)
                if (col[r] >= 0) sm.ref[mb][col[r]] = 1;
            __syncwarp();
            if (lane == 0) mbar_arrive(&sm.full_m[mb]);
            mb ^= 1;
            if (mb == 0) phm ^= 1;
            // per (row, slot): the slot's byte offset inside its row of a K-major
            // SW128 tile -- row n = kBRows bw + r at n * 128 B, 16-byte unit
            // (k / 4) ^ (n % 8) with n % 8 = r % 8 -- is the same in every chunk
            // (k = col - 32 c changes k / 4 by multiples of 8), so it is formed
            // once; packed with the slot's chunk (bits 16..) and the lo part
            int32_t pk[kBRows];
            float vlo[kBRows];
#pragma unroll
            for (int r = 0; r < kBRows; r++) {
                const int32_t k = col[r];
                pk[r] = k < 0 ? -1
                              : (r * 128 + (((((uint32_t)k >> 2) ^ (uint32_t)r) & 7u) << 4) + ((k & 3) << 2)) |
                                    ((k >> 5) << 16);
                vlo[r] = tf32_lo(val[r]);
            }
#ifdef LF_TC_TRACE
            if (lane == 0) atomicAdd(&lf_tc_trace[blockIdx.x][16], (unsigned long long)(clock64() - tb0));
#endif
            for (int c = 0; c < x.nch; c++) {
                TC_WAIT(6, &sm.empty_v[sv], phv ^ 1);
#ifdef LF_TC_TRACE
                const long long tc0 = clock64();
#endif
                // zero the warp's rows of the chunk (kBRows x 128 B per tile, 16 B per lane per store)
                char *th = reinterpret_cast<char *>(sm.vhi[sv]) + kBRows * bw * 128;
                char *tl = reinterpret_cast<char *>(sm.vlo[sv]) + kBRows * bw * 128;
#pragma unroll
                for (int u = 0; u < kBRows / 4; u++) {
                    *reinterpret_cast<float4 *>(th + (u * 32 + lane) * 16) = make_float4(0.f, 0.f, 0.f, 0.f);
                    *reinterpret_cast<float4 *>(tl + (u * 32 + lane) * 16) = make_float4(0.f, 0.f, 0.f, 0.f);
                }
                __syncwarp();
#pragma unroll
                for (int r = 0; r < kBRows; r++) {
                    if ((pk[r] >> 16) == c) {  // slot in this chunk (pk = -1: none)
                        const int o = pk[r] & 0xffff;
                        *reinterpret_cast<float *>(th + o) = val[r];
                        *reinterpret_cast<float *>(tl + o) = vlo[r];
                    }
                }
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> tensor core reads
                __syncwarp();
                if (lane == 0) mbar_arrive(&sm.full_v[sv]);
#ifdef LF_TC_TRACE
                if (lane == 0) atomicAdd(&lf_tc_trace[blockIdx.x][17], (unsigned long long)(clock64() - tc0));
#endif
                if (++sv == kTcVStages) {
                    sv = 0;
                    phv ^= 1;
                }
            }
        }
    } else if (warp == kWMma) {
        if (lane == 0) {
            // ===== MMA issuer (one thread) =====
            constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(kTcN >> 3) << 17) |
                                       ((uint32_t)(128 >> 4) << 24);  // F32 accum, TF32 A/B, K-major B, N, M = 128
            uint32_t sa = 0, pha = 0, sv = 0, phv = 0, d = 0, phd = 0;
            for (TcIter it(a); it.g < n_groups; it.next(a)) {
                const TcGroup &x = it.x;
                if (!x.mma) continue;
                TC_WAIT(7, &sm.empty_d[d], phd ^ 1);
                tc_fence_after();
                const uint32_t dcol = tmem + 128 * d;
                for (int c = 0; c < x.nch; c++) {
                    TC_WAIT(8, &sm.full_a[sa], pha);
                    TC_WAIT(9, &sm.full_v[sv], phv);
                    tc_fence_after();
                    const int nks = min(kTcK / 8, (x.span - kTcK * c + 7) / 8);
                    const uint64_t dh = sw128_desc(sm.vhi[sv]), dl = sw128_desc(sm.vlo[sv]);
                    const uint32_t a_raw = tmem + kColA + 64 * sa;
#ifdef LF_TC_TRACE
                    const long long tm0 = clock64();
#endif
                    for (int ks = 0; ks < nks; ks++) {
                        tc_mma(dcol, a_raw + 8 * ks, dh + 2 * ks, idesc, (c | ks) != 0);
                        tc_mma(dcol, a_raw + 32 + 8 * ks, dh + 2 * ks, idesc, 1);
                        tc_mma(dcol, a_raw + 8 * ks, dl + 2 * ks, idesc, 1);
                    }
#ifdef LF_TC_TRACE
                    atomicAdd(&lf_tc_trace[blockIdx.x][19], (unsigned long long)(clock64() - tm0));
#endif
                    tc_commit(&sm.empty_a[sa]);
                    tc_commit(&sm.empty_v[sv]);
                    if (++sa == kTcAStages) {
                        sa = 0;
                        pha ^= 1;
                    }
                    if (++sv == kTcVStages) {
                        sv = 0;
                        phv ^= 1;
                    }
                }
                tc_commit(&sm.full_d[d]);
                d ^= 1;
                if (d == 0) phd ^= 1;
            }
        }
    } else if (lane == 0) {
        // ===== TMA producer (one thread): each group's CELL rows, then its
        // B window in chunks of 32 rows, into their rings =====
        uint32_t sb = 0, phb = 0, sc = 0, phc = 0;
        const bool packed = a.ldb == a.J;
        for (TcIter it(a); it.g < n_groups; it.next(a)) {
            const TcGroup &x = it.x;
            if (!x.mma) continue;
            {
                const int64_t s0 = x.slot0 & ~int64_t(3);
                const int64_t s1 = (x.slot0 + ((int64_t)x.nr << x.t) + 3) & ~int64_t(3);
                const uint32_t bytes = (uint32_t)((s1 - s0) * 4);
                TC_WAIT(10, &sm.empty_c[sc], phc ^ 1);
                mbar_expect_tx(&sm.full_c[sc], 2 * bytes);
                bulk_g2s(sm.ccol[sc], a.col + s0, bytes, &sm.full_c[sc]);
                bulk_g2s(sm.cval[sc], a.val + s0, bytes, &sm.full_c[sc]);
                if (++sc == kTcCStages) {
                    sc = 0;
                    phc ^= 1;
                }
            }
            for (int c = 0; c < x.nch; c++) {
                const int kn = min(kTcK, x.span - kTcK * c);
                const uint32_t row_bytes = (uint32_t)a.J * 4;
                TC_WAIT(11, &sm.empty_b[sb], phb ^ 1);
                mbar_expect_tx(&sm.full_b[sb], row_bytes * kn);
                const float *src = a.B + (int64_t)(x.lo + kTcK * c) * a.ldb;
                if (packed) {
                    bulk_g2s(sm.bwin[sb], src, row_bytes * kn, &sm.full_b[sb]);
                } else {
                    for (int kk = 0; kk < kn; kk++)
                        bulk_g2s(sm.bwin[sb] + kk * a.J, src + (int64_t)kk * a.ldb, row_bytes, &sm.full_b[sb]);
                }
                if (++sb == kTcBStages) {
                    sb = 0;
                    phb ^= 1;
                }
            }
        }
    }
#ifdef LF_TC_TRACE
    if (lane == 0) atomicMax(&lf_tc_trace[blockIdx.x][12 + (warp < kWEpi ? 0 : warp < kWBuild ? 1 : warp < kWMma ? 2 : 3)],
                             (unsigned long long)(clock64() - t_start));
#endif
    tc_fence_before();
    __syncthreads();
    if (warp == kWMma) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(kTmemCols) : "memory");
    }
}

// Per group of kTcN CELL rows: window = [min first real column, max last real
// column] over its rows (columns are sorted within a CELL row, R6).  One
// 128-thread block per group, thread n reading row n (its real-slot count and
// two columns: every load of the group in flight at once), block min / max.
// (Folding this reduction into slot_fill with atomics measured slower: 181 ->
// 253-371 us on c3b, vs 40 us for this kernel.)
__global__ void __launch_bounds__(kTcN) tc_window_kernel(const BucketDev *__restrict__ bk, int nb, int64_t n_groups,
                                                         const int32_t *__restrict__ col,
                                                         const int32_t *__restrict__ src_cnt,
                                                         int2 *__restrict__ win) {
    __shared__ int smn[kTcN / 32], smx[kTcN / 32];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int64_t g = blockIdx.x; g < n_groups; g += gridDim.x) {
        int lo_b = 0, hi_b = nb - 1;  // bucket of group g
        while (lo_b < hi_b) {
            const int m = (lo_b + hi_b + 1) >> 1;
            if (__ldg(&bk[m].task_off) <= g) lo_b = m;
            else hi_b = m - 1;
        }
        const BucketDev &b = bk[lo_b];
        const int64_t r0 = (g - __ldg(&b.task_off)) * kTcN;
        const int n = threadIdx.x;
        int mn = INT32_MAX, mx = -1;
        if (r0 + n < __ldg(&b.n_rows_pad)) {
            const int cnt = __ldg(src_cnt + __ldg(&b.row_off) + r0 + n);
            if (cnt > 0) {
                const int64_t s = __ldg(&b.slot_off) + ((r0 + n) << __ldg(&b.t));
                mn = __ldg(col + s);
                mx = __ldg(col + s + cnt - 1);
            }
        }
        mn = __reduce_min_sync(kFull, mn);
        mx = __reduce_max_sync(kFull, mx);
        if (lane == 0) {
            smn[w] = mn;
            smx[w] = mx;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int q = 1; q < kTcN / 32; q++) {
                mn = min(mn, smn[q]);
                mx = max(mx, smx[q]);
            }
            win[g] = mx < 0 ? make_int2(0, 0) : make_int2(mn, mx - mn + 1);
        }
        __syncthreads();
    }
}

}  // namespace

cudaError_t launch_tc_windows(const BucketDev *bk_t, int nb_t, int64_t n_groups, const int32_t *col,
                              const int32_t *src_cnt, int2 *win, cudaStream_t s) {
    if (n_groups == 0) return cudaSuccess;
    const int grid = (int)std::min<int64_t>(n_groups, (int64_t)sm_count() * 64);
    tc_window_kernel<<<grid, kTcN, 0, s>>>(bk_t, nb_t, n_groups, col, src_cnt, win);
    return cudaGetLastError();
}

bool tc_ok(const SpmmArgs &a) {
    return a.tc && a.nb_t > 0 && a.tc_win && a.J >= 32 && a.J <= 128 && a.J % 4 == 0 && a.ldb % 4 == 0 &&
           a.ldc % 4 == 0 && ((uintptr_t)a.B & 15) == 0 && (a.c_bits & 15) == 0;
}

cudaError_t launch_cell_spmm_tc(const SpmmArgs &a, cudaStream_t s) {
    static int attr_set[64];
    const int dev = current_device();
    if (!attr_set[dev]) {
        cudaError_t e = cudaFuncSetAttribute(cell_spmm_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             (int)kTcSmem);
        if (e != cudaSuccess) return e;
        attr_set[dev] = 1;
    }
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((int64_t)sm_count(), a.n_groups_t));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(kTcWarps * 32);
    cfg.dynamicSmemBytes = kTcSmem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;  // overlap zero_rows_kernel
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
#ifndef LF_TC_TRACE
    return cudaLaunchKernelEx(&cfg, cell_spmm_tc_kernel, a);
#else
    static std::vector<unsigned long long> zero(1024 * 24, 0), h(1024 * 24);
    cudaMemcpyToSymbolAsync(lf_tc_trace, zero.data(), zero.size() * 8, 0, cudaMemcpyHostToDevice, s);
    cudaError_t e = cudaLaunchKernelEx(&cfg, cell_spmm_tc_kernel, a);
    cudaStreamSynchronize(s);
    cudaMemcpyFromSymbol(h.data(), lf_tc_trace, h.size() * 8);
    const char *names[24] = {"ld:full_m", "ld:full_b", "ld:empty_a", "ep:full_d", "bu:full_c", "bu:empty_m",
                             "bu:empty_v", "mma:empty_d", "mma:full_a", "mma:full_v", "tma:empty_c", "tma:empty_b",
                             "T:loaders", "T:epilogue", "T:builders", "T:mma/tma", "bu:extract", "bu:chunks",
                             "bu:tcgroup", "mma:issue", "ld:work", "x", "x", "x"};
    fprintf(stderr, "tc trace (grid %d, mean cycles per CTA):", grid);
    for (int k = 0; k < 21; k++) {
        double sum = 0;
        for (int b = 0; b < grid; b++) sum += (double)h[b * 24 + k];
        fprintf(stderr, " %s=%.0f", names[k], sum / grid);
    }
    fprintf(stderr, "\n");
    return e;
#endif
}

}  // namespace lf
