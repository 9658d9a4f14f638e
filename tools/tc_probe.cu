// tc_probe.cu -- checks the tcgen05 conventions cell_spmm_tc.cu relies on, on
// one 128 x N x 32 tile (kind::tf32, A in TMEM, B in smem K-major SW128):
//   1. layouts: D[m][n] = sum_k A[m][k] B[k][n] with A at TMEM lane m column k,
//      B[k][n] at (n/8)*1024 + (n%8)*128 + ((k/4) ^ (n%8))*16 + (k%4)*4,
//      D at TMEM lane m column n -- exact on small integers;
//   2. how the tensor core reads fp32 bits as tf32 (truncation or rounding);
//   3. the 3xTF32 split (hi = bits & 0xffffe000, lo = x - hi) error.
// nvcc -gencode arch=compute_100a,code=sm_100a -o tools/tc_probe tools/tc_probe.cu
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void st32(uint32_t t, const uint32_t (&r)[32]) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};"
        :: "r"(t), "r"(r[0]),"r"(r[1]),"r"(r[2]),"r"(r[3]),"r"(r[4]),"r"(r[5]),"r"(r[6]),"r"(r[7]),"r"(r[8]),"r"(r[9]),"r"(r[10]),"r"(r[11]),"r"(r[12]),"r"(r[13]),"r"(r[14]),"r"(r[15]),"r"(r[16]),"r"(r[17]),"r"(r[18]),"r"(r[19]),"r"(r[20]),"r"(r[21]),"r"(r[22]),"r"(r[23]),"r"(r[24]),"r"(r[25]),"r"(r[26]),"r"(r[27]),"r"(r[28]),"r"(r[29]),"r"(r[30]),"r"(r[31]) : "memory");
}
__device__ __forceinline__ void ld32(uint32_t t, uint32_t (&r)[32]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]),"=r"(r[1]),"=r"(r[2]),"=r"(r[3]),"=r"(r[4]),"=r"(r[5]),"=r"(r[6]),"=r"(r[7]),"=r"(r[8]),"=r"(r[9]),"=r"(r[10]),"=r"(r[11]),"=r"(r[12]),"=r"(r[13]),"=r"(r[14]),"=r"(r[15]),"=r"(r[16]),"=r"(r[17]),"=r"(r[18]),"=r"(r[19]),"=r"(r[20]),"=r"(r[21]),"=r"(r[22]),"=r"(r[23]),"=r"(r[24]),"=r"(r[25]),"=r"(r[26]),"=r"(r[27]),"=r"(r[28]),"=r"(r[29]),"=r"(r[30]),"=r"(r[31]) : "r"(t));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void mma(uint32_t d, uint32_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
    asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], [%1], %2, %3, p;\n}"
                 :: "r"(d), "r"(a), "l"(b), "r"(idesc), "r"(acc) : "memory");
}
__device__ __forceinline__ uint32_t hi_bits(float x) { return __float_as_uint(x) & 0xffffe000u; }

constexpr int N = 128;
// mode 0: one MMA chain with raw fp32 bits; 1: 3xTF32 split
__global__ void probe(const float *A, const float *B, float *D, int mode) {
    __shared__ __align__(1024) float bt[2][N * 32];  // raw/hi, lo
    __shared__ uint32_t tbase;
    __shared__ __align__(8) uint64_t bar;
    const int tid = threadIdx.x, warp = tid >> 5;
    for (int q = tid; q < N * 32; q += blockDim.x) {
        const int n = q / 32, k = q % 32;
        const float x = B[k * N + n];
        const int off = (n / 8) * 256 + (n % 8) * 32 + (((k / 4) ^ (n % 8)) * 4) + (k % 4);
        const float h = __uint_as_float(hi_bits(x));
        bt[0][off] = mode ? h : x;
        bt[1][off] = x - h;
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" :: "r"(smem_u32(&tbase)), "r"(512));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 0) asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(&bar)), "r"(1));
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t t = tbase;
    // A: thread m (lane m) writes row m: cols [256, 288) raw/hi, [288, 320) lo
    uint32_t r[32], rl[32];
    for (int k = 0; k < 32; k++) {
        const float x = A[tid * 32 + k];
        const uint32_t h = hi_bits(x);
        r[k] = mode ? h : __float_as_uint(x);
        rl[k] = __float_as_uint(x - __uint_as_float(h));
    }
    st32(t + ((uint32_t)(warp * 32) << 16) + 256, r);
    st32(t + ((uint32_t)(warp * 32) << 16) + 288, rl);
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (tid == 0) {
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(N >> 3) << 17) | (8u << 24);
        for (int ks = 0; ks < 4; ks++) {
            for (int part = 0; part < (mode ? 3 : 1); part++) {
                const int bi = part == 2 ? 1 : 0;           // hi.hi, lo(A).hi(B), hi(A).lo(B)
                const uint32_t a = t + 256 + (part == 1 ? 32 : 0) + ks * 8;
                const uint64_t addr = smem_u32(&bt[bi][0]) + ks * 32;
                const uint64_t desc = ((addr >> 4) & 0x3FFF) | (1ull << 16) | (64ull << 32) | (1ull << 46) | (2ull << 61);
                mma(t, a, desc, idesc, (ks | part) != 0);
            }
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" :: "r"(smem_u32(&bar)) : "memory");
    }
    asm volatile("{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}" :: "r"(smem_u32(&bar)), "r"(0) : "memory");
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    for (int c = 0; c < N; c += 32) {
        ld32(t + ((uint32_t)(warp * 32) << 16) + c, r);
        for (int i = 0; i < 32; i++) D[tid * N + c + i] = __uint_as_float(r[i]);
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" :: "r"(t), "r"(512));
}

static float trunc_tf32(float x) { uint32_t u; memcpy(&u, &x, 4); u &= 0xffffe000u; float y; memcpy(&y, &u, 4); return y; }
static float rn_tf32(float x) { uint32_t u; memcpy(&u, &x, 4); u += 0x1000u + ((u >> 13) & 1); u &= 0xffffe000u; float y; memcpy(&y, &u, 4); return y; }

int main() {
    std::vector<float> A(128 * 32), B(32 * N), D(128 * N);
    float *dA, *dB, *dD;
    CK(cudaMalloc(&dA, A.size() * 4)); CK(cudaMalloc(&dB, B.size() * 4)); CK(cudaMalloc(&dD, D.size() * 4));
    srand(1);
    // 1. layout: integers
    for (auto &x : A) x = (float)(rand() % 7 - 3);
    for (auto &x : B) x = (float)(rand() % 31 - 15);
    for (int mode = 0; mode < 2; mode++) {
        CK(cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice));
        probe<<<1, 128>>>(dA, dB, dD, mode);
        CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost));
        int bad = 0;
        for (int m = 0; m < 128; m++)
            for (int n = 0; n < N; n++) {
                double s = 0;
                for (int k = 0; k < 32; k++) s += (double)A[m * 32 + k] * B[k * N + n];
                if ((double)D[m * N + n] != s) { if (bad < 5) printf("int mode %d: D[%d][%d] = %g, want %g\n", mode, m, n, D[m * N + n], s); bad++; }
            }
        printf("layout check (integers, mode %d): %s (%d mismatches)\n", mode, bad ? "FAIL" : "ok", bad);
    }
    // 2. tf32 conversion semantics and 3. 3xTF32 error
    for (auto &x : A) x = (float)((rand() & 0xffffff) * 0x1p-23 - 1.0);
    for (auto &x : B) x = (float)((rand() & 0xffffff) * 0x1p-23 - 1.0);
    CK(cudaMemcpy(dA, A.data(), A.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice));
    for (int mode = 0; mode < 2; mode++) {
        probe<<<1, 128>>>(dA, dB, dD, mode);
        CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(D.data(), dD, D.size() * 4, cudaMemcpyDeviceToHost));
        double e_tr = 0, e_rn = 0, e_ex = 0;
        for (int m = 0; m < 128; m++)
            for (int n = 0; n < N; n++) {
                double st = 0, sr = 0, se = 0, sa = 0;
                for (int k = 0; k < 32; k++) {
                    const float a = A[m * 32 + k], b = B[k * N + n];
                    st += (double)trunc_tf32(a) * trunc_tf32(b);
                    sr += (double)rn_tf32(a) * rn_tf32(b);
                    se += (double)a * b;
                    sa += fabs((double)a * b);
                }
                const double d = D[m * N + n];
                e_tr = fmax(e_tr, fabs(d - st) / sa);
                e_rn = fmax(e_rn, fabs(d - sr) / sa);
                e_ex = fmax(e_ex, fabs(d - se) / sa);
            }
        printf("mode %d (%s): max rel err vs trunc-tf32 %.3g, vs rn-tf32 %.3g, vs exact %.3g\n", mode,
               mode ? "3xTF32 split" : "raw fp32 bits", e_tr, e_rn, e_ex);
    }
    return 0;
}
