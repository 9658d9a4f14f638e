// gather_roofline.cu -- B200 microbenchmark: random row gathers from a dense
// fp32 table (the B operand of SpMM), to measure the L2/L1 -> SM gather
// bandwidth that bounds a CELL SpMM whose B is gathered row by row.
//   ./gather_roofline  (prints one line per (table MB, row bytes, mode))
// Each warp loads one random row of `row_bytes` per step (lanes x float4),
// U rows in flight per warp; indices come from a precomputed random array
// (streamed, 4 B per row).  GB/s counts row bytes delivered to the SMs.
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

template <int NV, int U, bool L1>
__global__ void __launch_bounds__(256) gather(const float4 *__restrict__ tab, const int *__restrict__ idx, int64_t n_idx,
                                              int row_f4, float4 *__restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = (gridDim.x * (int64_t)blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  for (int64_t q = w * 32; q < n_idx; q += nw * 32) {
    int my = q + lane < n_idx ? idx[q + lane] : 0;
    #pragma unroll
    for (int s = 0; s < 32; s += U) {
      float4 v[U][NV];
      #pragma unroll
      for (int u = 0; u < U; u++) {
        int r = __shfl_sync(0xffffffffu, my, s + u);
        #pragma unroll
        for (int m = 0; m < NV; m++) {
          const float4 *p = tab + (int64_t)r * row_f4 + m * 32 + lane;
          if (L1) v[u][m] = __ldg(p);
          else {
            float4 t; asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(t.x), "=f"(t.y), "=f"(t.z), "=f"(t.w) : "l"(p));
            v[u][m] = t;
          }
        }
      }
      #pragma unroll
      for (int u = 0; u < U; u++)
        #pragma unroll
        for (int m = 0; m < NV; m++) { acc.x += v[u][m].x; acc.y += v[u][m].y; acc.z += v[u][m].z; acc.w += v[u][m].w; }
    }
  }
  if (acc.x + acc.y + acc.z + acc.w == 12345.f) out[0] = acc;
}

template <int NV, int U, bool L1>
double run(const float4 *tab, const int *idx, int64_t n_idx, float4 *out, int blocks) {
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  gather<NV, U, L1><<<blocks, 256>>>(tab, idx, n_idx, NV * 32, out);
  CK(cudaEventRecord(a));
  const int it = 5;
  for (int i = 0; i < it; i++) gather<NV, U, L1><<<blocks, 256>>>(tab, idx, n_idx, NV * 32, out);
  CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return (double)n_idx * NV * 512 * it / (ms * 1e-3) / 1e9;
}

int main() {
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const int64_t n_idx = 32 << 20;  // 32M row gathers per launch
  int *idx; CK(cudaMalloc(&idx, n_idx * 4));
  float4 *out; CK(cudaMalloc(&out, 64));
  const int64_t max_bytes = 1LL << 30;
  float4 *tab; CK(cudaMalloc(&tab, max_bytes));
  CK(cudaMemset(tab, 0, max_bytes));
  std::vector<int> h(n_idx);
  printf("{\"sms\": %d}\n", sms);
  for (int64_t mb : {4, 16, 32, 48, 96, 256, 1024}) {
    for (int row_bytes : {512, 1024}) {
      const int64_t rows = mb * (1LL << 20) / row_bytes;
      uint64_t s = 88172645463325252ull;
      for (int64_t i = 0; i < n_idx; i++) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = (int)(s % rows); }
      CK(cudaMemcpy(idx, h.data(), n_idx * 4, cudaMemcpyHostToDevice));
      for (int occ : {4, 8}) {
        const int blocks = sms * occ;
        double g1, g2;
        if (row_bytes == 512) { g1 = run<1, 8, true>(tab, idx, n_idx, out, blocks); g2 = run<1, 8, false>(tab, idx, n_idx, out, blocks); }
        else { g1 = run<2, 4, true>(tab, idx, n_idx, out, blocks); g2 = run<2, 4, false>(tab, idx, n_idx, out, blocks); }
        printf("{\"table_mb\": %lld, \"row_bytes\": %d, \"blocks_per_sm\": %d, \"gbs_l1\": %.0f, \"gbs_nol1\": %.0f}\n",
               (long long)mb, row_bytes, occ, g1, g2);
      }
    }
  }
  return 0;
}
