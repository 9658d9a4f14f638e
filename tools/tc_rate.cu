// tc_rate.cu -- tcgen05.mma kind::tf32 issue rate on one SM: n_mma MMAs into
// one accumulator (M = 128, K = 8), A from TMEM ("TS") or from shared memory
// ("SS"), N in {32, 64, 128, 256}; clock64 around issue -> commit -> wait.
// nvcc -gencode arch=compute_100a,code=sm_100a -o tools/tc_rate tools/tc_rate.cu
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <bool TS>
__global__ void rate(int n_mma, int N, long long *out) {
    extern __shared__ __align__(1024) uint8_t sm_raw[];
    float *tile = reinterpret_cast<float *>((reinterpret_cast<uintptr_t>(sm_raw) + 1023) & ~uintptr_t(1023));
    __shared__ uint32_t tbase;
    __shared__ __align__(8) uint64_t bar;
    for (int i = threadIdx.x; i < 256 * 32 * 2; i += blockDim.x) tile[i] = 1.0f;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tbase)), "r"(512));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&bar)), "r"(1));
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (threadIdx.x == 0) {
        const uint32_t t = tbase;
        const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | (8u << 24);
        const uint64_t b_addr = smem_u32(tile);
        const uint64_t bdesc = ((b_addr >> 4) & 0x3FFF) | (1ull << 16) | (64ull << 32) | (1ull << 46) | (2ull << 61);
        const uint64_t a_addr = smem_u32(tile + 256 * 32);
        const uint64_t adesc = ((a_addr >> 4) & 0x3FFF) | (1ull << 16) | (64ull << 32) | (1ull << 46) | (2ull << 61);
        long long t0 = clock64();
        for (int i = 0; i < n_mma; i++) {
            const uint32_t acc = i > 0;
            if (TS)
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}"
                             ::"r"(t), "r"(t + 256 + 8 * (i & 3)), "l"(bdesc + 2 * (i & 3)), "r"(idesc), "r"(acc));
            else
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}"
                             ::"r"(t), "l"(adesc + 2 * (i & 3)), "l"(bdesc + 2 * (i & 3)), "r"(idesc), "r"(acc));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)) : "memory");
        asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}" ::"r"(smem_u32(&bar)), "r"(0) : "memory");
        long long t1 = clock64();
        out[0] = t1 - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase), "r"(512));
}

// the cell_spmm_tc issue pattern: per chunk 4 k-steps x 3 MMAs (A raw/lo from a
// 4-slot TMEM ring, B hi/lo from a 3-slot smem ring), 2 commits per chunk,
// D alternating between 2 accumulators every 5 chunks
__global__ void pattern(int n_chunks, int commits, long long *out) {
    extern __shared__ __align__(1024) uint8_t sm_raw[];
    float *tile = reinterpret_cast<float *>(sm_raw);
    __shared__ uint32_t tbase;
    __shared__ __align__(8) uint64_t bar[2];
    for (int i = threadIdx.x; i < 6 * 128 * 32; i += blockDim.x) tile[i] = 1.0f;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tbase)), "r"(512));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&bar[0])), "r"(1));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&bar[1])), "r"(1));
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (threadIdx.x == 0) {
        const uint32_t t = tbase;
        const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(128 >> 3) << 17) | (8u << 24);
        long long t0 = clock64();
        for (int c = 0; c < n_chunks; c++) {
            const int sa = c & 3, sv = c % 3, d = (c / 5) & 1;
            const uint64_t ah = smem_u32(tile + (2 * sv) * 128 * 32), al = smem_u32(tile + (2 * sv + 1) * 128 * 32);
            const uint64_t dh = ((ah >> 4) & 0x3FFF) | (1ull << 16) | (64ull << 32) | (1ull << 46) | (2ull << 61);
            const uint64_t dl = ((al >> 4) & 0x3FFF) | (1ull << 16) | (64ull << 32) | (1ull << 46) | (2ull << 61);
            const uint32_t a_raw = t + 256 + 64 * sa, dcol = t + 128 * d;
            if (commits == 2) asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            for (int ks = 0; ks < 4; ks++) {
                const uint32_t acc = (c % 5 | ks) != 0;
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}"
                             ::"r"(dcol), "r"(a_raw + 8 * ks), "l"(dh + 2 * ks), "r"(idesc), "r"(acc));
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}"
                             ::"r"(dcol), "r"(a_raw + 32 + 8 * ks), "l"(dh + 2 * ks), "r"(idesc), "r"(1u));
                asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}"
                             ::"r"(dcol), "r"(a_raw + 8 * ks), "l"(dl + 2 * ks), "r"(idesc), "r"(1u));
            }
            if (commits >= 1) {
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar[1])) : "memory");
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar[1])) : "memory");
            }
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar[0])) : "memory");
        asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}" ::"r"(smem_u32(&bar[0])), "r"(0) : "memory");
        long long t1 = clock64();
        out[0] = t1 - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase), "r"(512));
}

int main() {
    long long *d, h;
    cudaMalloc(&d, 8);
    const int smem = 256 * 32 * 2 * 4 + 1024;
    cudaFuncSetAttribute(rate<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(rate<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int ts = 1; ts >= 0; ts--)
        for (int N : {32, 64, 128, 256}) {
            for (int n : {64, 1024}) {
                if (ts) rate<true><<<1, 128, smem>>>(n, N, d);
                else rate<false><<<1, 128, smem>>>(n, N, d);
                cudaError_t e = cudaDeviceSynchronize();
                cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
                printf("%s N=%3d n_mma=%5d: %8lld clk  %.1f clk/mma (floor N/2 = %d)  %s\n", ts ? "TS" : "SS", N, n, h,
                       (double)h / n, N / 2, cudaGetErrorString(e));
            }
        }
    const int psmem = 6 * 128 * 32 * 4;
    cudaFuncSetAttribute(pattern, cudaFuncAttributeMaxDynamicSharedMemorySize, psmem);
    for (int commits = 0; commits < 3; commits++) {
        pattern<<<1, 128, psmem>>>(500, commits, d);
        cudaError_t e = cudaDeviceSynchronize();
        cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
        printf("pattern (commits %d): %.1f clk/mma  %s\n", commits, (double)h / (500 * 12), cudaGetErrorString(e));
        pattern<<<148, 128, psmem>>>(500, commits, d);
        e = cudaDeviceSynchronize();
        cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
        printf("pattern x148 CTAs (commits %d): %.1f clk/mma  %s\n", commits, (double)h / (500 * 12), cudaGetErrorString(e));
    }
    return 0;
}
