// gather4_replay.cu -- B200 microbenchmark: replay a matrix's column sequence
// as B-row gathers done by the TMA engine with sm_100's 2-D tensor gather
// (cp.async.bulk.tensor.2d.tile::gather4: 4 rows of 512 B per instruction,
// landing in shared memory, completion on an mbarrier), read back by consumer
// warps with LDS.128.  Compared with tools/gather_replay.cu (LDG gathers into
// registers), the rows in flight live in shared memory, not registers.
//   ./gather4_replay cols.bin n_cols
// One producer warp per block (lane q issues gather4 q of a stage), NC
// consumer warps; a stage of R rows is consumed by one warp.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, int n) {
  asm volatile("mbarrier.init.shared.b64 [%0], %1;" ::"r"(sa(b)), "r"(n));
}
__device__ __forceinline__ bool mbar_try(uint64_t *b, int ph) {
  uint32_t ok;
  asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
               : "=r"(ok) : "r"(sa(b)), "r"(ph) : "memory");
  return ok;
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, int ph) { while (!mbar_try(b, ph)) {} }
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
  asm volatile("mbarrier.arrive.shared.b64 _, [%0];" ::"r"(sa(b)) : "memory");
}
__device__ __forceinline__ void mbar_expect(uint64_t *b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void gather4(void *dst, const CUtensorMap *tm, int4 r, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(sa(dst)),
      "l"(tm), "r"(0), "r"(r.x), "r"(r.y), "r"(r.z), "r"(r.w), "r"(sa(bar))
      : "memory");
}

template <int R, int S, int NC>
__global__ void __launch_bounds__((NC + 1) * 32) replay_g4(const __grid_constant__ CUtensorMap tm,
                                                           const int *__restrict__ idx, int64_t n_idx,
                                                           float *__restrict__ out) {
  extern __shared__ __align__(1024) unsigned char sm[];
  float4 *buf = reinterpret_cast<float4 *>(sm);
  uint64_t *full = reinterpret_cast<uint64_t *>(sm + (size_t)S * R * 512), *empty = full + S;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; s++) { mbar_init(full + s, 1); mbar_init(empty + s, 1); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int64_t n_st = n_idx / R;
  const int64_t per = (n_st + gridDim.x - 1) / gridDim.x;
  const int64_t k0 = blockIdx.x * per, k1 = min(n_st, k0 + per);
  if (w == NC) {  // producer
    for (int64_t k = k0; k < k1; k++) {
      const int64_t j = k - k0;
      const int s = (int)(j % S);
      if (j >= S) mbar_wait(empty + s, (int)(((j / S) - 1) & 1));
      if (lane == 0) mbar_expect(full + s, R * 512);
      __syncwarp();
      if (lane < R / 4) {
        const int4 r = __ldcs(reinterpret_cast<const int4 *>(idx + k * R) + lane);
        gather4(buf + ((size_t)s * R + lane * 4) * 32, &tm, r, full + s);
      }
    }
    return;
  }
  float4 acc = make_float4(0, 0, 0, 0);
  for (int64_t k = k0 + w; k < k1; k += NC) {
    const int64_t j = k - k0;
    const int s = (int)(j % S);
    mbar_wait(full + s, (int)((j / S) & 1));
#pragma unroll 8
    for (int r = 0; r < R; r++) {
      const float4 v = buf[((size_t)s * R + r) * 32 + lane];
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(empty + s);
  }
  if (lane == 0) out[(int64_t)blockIdx.x * NC + w] = acc.x;
}

static PFN_cuTensorMapEncodeTiled_v12000 encode() {
  void *fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q));
  return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
}

template <int R, int S, int NC>
float run(const CUtensorMap &tm, const int *idx, int64_t n, float *out, int bps, int sms, std::vector<int> &h,
          const std::vector<float> &tabcol0) {
  const size_t smem = (size_t)S * R * 512 + 2 * S * 8;
  auto fn = replay_g4<R, S, NC>;
  CK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  const int grid = sms * bps;
  CK(cudaMemset(out, 0, (size_t)grid * NC * 4));
  fn<<<grid, (NC + 1) * 32, smem>>>(tm, idx, n, out);
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  // check: lane 0's column-0 sums of all rows of the covered stages
  std::vector<float> o((size_t)grid * NC);
  CK(cudaMemcpy(o.data(), out, o.size() * 4, cudaMemcpyDeviceToHost));
  double got = 0, want = 0;
  for (float x : o) got += x;
  for (int64_t q = 0; q < (n / R) * R; q++) want += tabcol0[h[q]];
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  CK(cudaEventRecord(a));
  const int it = 10;
  for (int i = 0; i < it; i++) fn<<<grid, (NC + 1) * 32, smem>>>(tm, idx, n, out);
  CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  ms /= it;
  printf("{\"R\": %d, \"S\": %d, \"NC\": %d, \"blocks_per_sm\": %d, \"smem_kb\": %.0f, \"ms\": %.4f, \"gbs\": %.0f, \"check\": %s}\n",
         R, S, NC, bps, smem / 1024.0, ms, (double)(n / R) * R * 512 / (ms * 1e-3) / 1e9, got == want ? "true" : "false");
  fflush(stdout);
  return ms;
}

int main(int argc, char **argv) {
  if (argc < 3) { printf("usage: gather4_replay cols.bin n_cols\n"); return 1; }
  FILE *f = fopen(argv[1], "rb");
  if (!f) { printf("cannot open %s\n", argv[1]); return 1; }
  fseek(f, 0, SEEK_END); const int64_t n = ftell(f) / 4; fseek(f, 0, SEEK_SET);
  std::vector<int> h(n);
  if ((int64_t)fread(h.data(), 4, n, f) != n) { printf("short read\n"); return 1; }
  fclose(f);
  const int64_t K = atoll(argv[2]);
  const int J = 128;
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  int *idx; CK(cudaMalloc(&idx, n * 4));
  CK(cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice));
  std::vector<float> ht((size_t)K * J), col0(K);
  for (int64_t r = 0; r < K; r++) {
    col0[r] = (float)(r % 7);
    for (int j = 0; j < J; j++) ht[(size_t)r * J + j] = (float)((r + j) % 7);
  }
  float *tab; CK(cudaMalloc(&tab, (size_t)K * J * 4));
  CK(cudaMemcpy(tab, ht.data(), ht.size() * 4, cudaMemcpyHostToDevice));
  float *out; CK(cudaMalloc(&out, (size_t)sms * 8 * 32 * 4));
  CUtensorMap tm;
  cuuint64_t gdim[2] = {(cuuint64_t)J, (cuuint64_t)K};
  cuuint64_t gstr[1] = {(cuuint64_t)J * 4};
  cuuint32_t box[2] = {(cuuint32_t)J, 1};
  cuuint32_t es[2] = {1, 1};
  CUresult cr = encode()(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, tab, gdim, gstr, box, es,
                         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                         CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (cr != CUDA_SUCCESS) { printf("tensor map encode failed %d\n", (int)cr); return 1; }
  run<16, 8, 4>(tm, idx, n, out, 1, sms, h, col0);
  run<16, 12, 8>(tm, idx, n, out, 1, sms, h, col0);
  run<16, 24, 8>(tm, idx, n, out, 1, sms, h, col0);
  run<32, 12, 8>(tm, idx, n, out, 1, sms, h, col0);
  run<32, 6, 4>(tm, idx, n, out, 2, sms, h, col0);
  run<16, 12, 4>(tm, idx, n, out, 2, sms, h, col0);
  run<8, 24, 4>(tm, idx, n, out, 2, sms, h, col0);
  run<8, 48, 8>(tm, idx, n, out, 1, sms, h, col0);
  run<64, 6, 8>(tm, idx, n, out, 1, sms, h, col0);
  return 0;
}
