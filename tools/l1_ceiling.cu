// l1_ceiling.cu -- B200 microbenchmark: what bounds the SpMM's B-row gathers
// per SM.  Random 512-B row gathers (J = 128 fp32) from a table of T bytes,
// delivered to registers by
//   v4  : LDG.128, one row per warp instruction (lanes x float4), U rows in flight
//   v8  : LDG.256 (ld.global.nc.v8.f32, sm_100+), two rows per warp instruction
//         (16 lanes x 8 floats each), U/2 instructions in flight
//   lds : the table staged once in shared memory (T <= 128 KB), LDS.128 gathers
// GB/s = row bytes delivered.  T = 64 KB..1 GB spans L1-, L2- and HBM-resident.
//   ./l1_ceiling
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ void ld8(const float *p, float (&a)[8]) {
  asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(a[0]), "=f"(a[1]), "=f"(a[2]), "=f"(a[3]), "=f"(a[4]), "=f"(a[5]), "=f"(a[6]), "=f"(a[7])
               : "l"(p));
}

template <int MODE, int U>
__global__ void __launch_bounds__(256) gather(const float *__restrict__ tab, int64_t rows, const int *__restrict__ idx,
                                              int64_t n_idx, float *__restrict__ out) {
  extern __shared__ __align__(16) float sm[];
  const int lane = threadIdx.x & 31;
  if (MODE == 2) {
    for (int64_t i = threadIdx.x; i < rows * 128; i += blockDim.x) sm[i] = tab[i];
    __syncthreads();
  }
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = (gridDim.x * (int64_t)blockDim.x) >> 5;
  float acc = 0.f;
  for (int64_t q = w * 32; q < n_idx; q += nw * 32) {
    const int my = q + lane < n_idx ? __ldcs(idx + q + lane) : 0;
    if (MODE == 1) {
      // two rows per instruction: lanes 0-15 row s+2u, lanes 16-31 row s+2u+1
#pragma unroll
      for (int s = 0; s < 32; s += 2 * U) {
        float v[U][8];
#pragma unroll
        for (int u = 0; u < U; u++) {
          const int r = __shfl_sync(0xffffffffu, my, s + 2 * u + (lane >> 4));
          ld8(tab + (int64_t)r * 128 + (lane & 15) * 8, v[u]);
        }
#pragma unroll
        for (int u = 0; u < U; u++)
#pragma unroll
          for (int e = 0; e < 8; e++) acc += v[u][e];
      }
    } else {
#pragma unroll
      for (int s = 0; s < 32; s += U) {
        float4 v[U];
#pragma unroll
        for (int u = 0; u < U; u++) {
          const int r = __shfl_sync(0xffffffffu, my, s + u);
          if (MODE == 0) v[u] = __ldg(reinterpret_cast<const float4 *>(tab + (int64_t)r * 128) + lane);
          else v[u] = reinterpret_cast<const float4 *>(sm + r * 128)[lane];
        }
#pragma unroll
        for (int u = 0; u < U; u++) acc += v[u].x + v[u].y + v[u].z + v[u].w;
      }
    }
  }
  if (acc == 12345.f) out[0] = acc;
}

template <int MODE, int U>
double run(const float *tab, int64_t rows, const int *idx, int64_t n, float *out, int blocks, size_t smem) {
  if (smem) CK(cudaFuncSetAttribute(gather<MODE, U>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a));
  CK(cudaEventCreate(&b));
  gather<MODE, U><<<blocks, 256, smem>>>(tab, rows, idx, n, out);
  CK(cudaGetLastError());
  CK(cudaEventRecord(a));
  const int it = 5;
  for (int i = 0; i < it; i++) gather<MODE, U><<<blocks, 256, smem>>>(tab, rows, idx, n, out);
  CK(cudaEventRecord(b));
  CK(cudaEventSynchronize(b));
  float ms;
  CK(cudaEventElapsedTime(&ms, a, b));
  return (double)n * 512 * it / (ms * 1e-3) / 1e9;
}

int main() {
  int sms;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int64_t n_idx = 32 << 20;
  int *idx;
  CK(cudaMalloc(&idx, n_idx * 4));
  float *out;
  CK(cudaMalloc(&out, 64));
  const int64_t max_bytes = 1LL << 30;
  float *tab;
  CK(cudaMalloc(&tab, max_bytes));
  CK(cudaMemset(tab, 0, max_bytes));
  std::vector<int> h(n_idx);
  for (int64_t kb : {64, 128, 1024, 4096, 65536, 1048576}) {
    const int64_t rows = kb * 1024 / 512;
    uint64_t s = 88172645463325252ull;
    for (int64_t i = 0; i < n_idx; i++) {
      s ^= s << 13;
      s ^= s >> 7;
      s ^= s << 17;
      h[i] = (int)(s % rows);
    }
    CK(cudaMemcpy(idx, h.data(), n_idx * 4, cudaMemcpyHostToDevice));
    for (int occ : {4, 8}) {
      const int blocks = sms * occ;
      const double v4 = run<0, 8>(tab, rows, idx, n_idx, out, blocks, 0);
      const double v8 = run<1, 4>(tab, rows, idx, n_idx, out, blocks, 0);
      const double v8d = run<1, 8>(tab, rows, idx, n_idx, out, blocks, 0);
      double lds = 0;
      if (kb <= 64 && occ == 4) lds = run<2, 8>(tab, rows, idx, n_idx, out, sms * 3, kb * 1024);
      printf("{\"table_kb\": %lld, \"blocks_per_sm\": %d, \"gbs_v4_u8\": %.0f, \"gbs_v8_u4\": %.0f, \"gbs_v8_u8\": %.0f, "
             "\"gbs_lds_3blk\": %.0f}\n",
             (long long)kb, occ, v4, v8, v8d, lds);
    }
  }
  return 0;
}
