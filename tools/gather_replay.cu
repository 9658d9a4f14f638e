// gather_replay.cu -- B200 microbenchmark: replay a real matrix's column
// sequence as B-row gathers (the SpMM's dominant traffic) with no index
// decoding, shuffles or C writes, to bound what the CELL SpMM kernel can reach
// on that matrix's access pattern at a given gather depth.
//   ./gather_replay cols.bin n_cols J
// cols.bin: int32 column indices in processing order (e.g. CSR order).
// Each warp takes 32 consecutive indices, gathers U rows at a time
// (lanes x float4 cover J = 128 floats per row), and sums them.
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

// ILV = 0: each warp replays a contiguous range of 32-index chunks (like the
// SpMM's per-warp claims); ILV = 1: each BLOCK takes a contiguous range and
// its 8 warps interleave over it (chunk start + w, start + w + 8, ...), so
// consecutive chunks -- consecutive rows -- are gathered on one SM at once
template <int U, int MODE, int ILV = 0>
__global__ void __launch_bounds__(256) replay(const float4 *__restrict__ tab, const int *__restrict__ idx, int64_t n_idx,
                                              int row_f4, float4 *__restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = (gridDim.x * (int64_t)blockDim.x) >> 5;
  float4 acc = make_float4(0, 0, 0, 0);
  const int64_t n_ch = (n_idx + 31) / 32;
  int64_t c_beg, c_end, c_step;
  if (ILV) {
    const int64_t wpb = blockDim.x >> 5, per = (n_ch + gridDim.x - 1) / gridDim.x;
    c_beg = blockIdx.x * per + (threadIdx.x >> 5);
    c_end = min(n_ch, (int64_t)(blockIdx.x + 1) * per);
    c_step = wpb;
  } else {
    const int64_t per = (n_ch + nw - 1) / nw;
    c_beg = w * per;
    c_end = min(n_ch, (w + 1) * per);
    c_step = 1;
  }
  for (int64_t ch = c_beg; ch < c_end; ch += c_step) {
    const int64_t q = ch * 32;
    int my = q + lane < n_idx ? __ldcs(idx + q + lane) : 0;
#pragma unroll
    for (int s = 0; s < 32; s += U) {
      float4 v[U];
#pragma unroll
      for (int u = 0; u < U; u++) {
        const int r = __shfl_sync(0xffffffffu, my, s + u);
        const float4 *p = tab + (int64_t)r * row_f4 + lane;
        if (MODE == 0) v[u] = __ldg(p);
        else {
          float4 t;
          asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(t.x), "=f"(t.y), "=f"(t.z), "=f"(t.w) : "l"(p));
          v[u] = t;
        }
      }
#pragma unroll
      for (int u = 0; u < U; u++) { acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w; }
    }
  }
  if (acc.x + acc.y + acc.z + acc.w == 12345.f) out[0] = acc;
}

template <int U, int MODE, int ILV = 0>
float run(const float4 *tab, const int *idx, int64_t n, int row_f4, float4 *out, int blocks) {
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  replay<U, MODE, ILV><<<blocks, 256>>>(tab, idx, n, row_f4, out);
  CK(cudaEventRecord(a));
  const int it = 10;
  for (int i = 0; i < it; i++) replay<U, MODE, ILV><<<blocks, 256>>>(tab, idx, n, row_f4, out);
  CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return ms / it;
}

// TMA variant: every lane of a warp issues one cp.async.bulk (a whole 512-B
// row, no registers held while in flight) into a per-warp 2-stage smem ring;
// completion through one mbarrier per stage (ROWS arrivals + tx bytes); the
// warp then reads each row with LDS.128 and refills the stage.
__device__ __forceinline__ void mbar_init(uint64_t *b, int n) {
  asm volatile("mbarrier.init.shared.b64 [%0], %1;" :: "r"((uint32_t)__cvta_generic_to_shared(b)), "r"(n));
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, int phase) {
  asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared.b64 p, [%0], %1;\n @!p bra W;\n}\n"
               :: "r"((uint32_t)__cvta_generic_to_shared(b)), "r"(phase) : "memory");
}
__device__ __forceinline__ void bulk_row(void *dst, const void *src, uint64_t *b) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(dst), m = (uint32_t)__cvta_generic_to_shared(b);
  asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], 512;" :: "r"(m) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], 512, [%2];"
               :: "r"(d), "l"(src), "r"(m) : "memory");
}

template <int ROWS, int WPB>
__global__ void __launch_bounds__(WPB * 32) replay_tma(const float4 *__restrict__ tab, const int *__restrict__ idx,
                                                        int64_t n_idx, float4 *__restrict__ out) {
  extern __shared__ __align__(128) unsigned char sm[];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  float4 *buf = reinterpret_cast<float4 *>(sm) + (size_t)w * 2 * ROWS * 32;
  uint64_t *bar = reinterpret_cast<uint64_t *>(sm + (size_t)WPB * 2 * ROWS * 512) + 2 * w;
  if (lane == 0) { mbar_init(bar, ROWS); mbar_init(bar + 1, ROWS); }
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const int64_t gw = (int64_t)blockIdx.x * WPB + w, nw = (int64_t)gridDim.x * WPB;
  const int64_t n_ch = n_idx / ROWS;
  const int64_t per = (n_ch + nw - 1) / nw;
  const int64_t c0 = gw * per, c1 = min(n_ch, c0 + per);
  float4 acc = make_float4(0, 0, 0, 0);
  auto issue = [&](int st, int64_t c) {
    if (c < c1 && lane < ROWS) {
      const int r = __ldcs(idx + c * ROWS + lane);
      bulk_row(buf + ((size_t)st * ROWS + lane) * 32, tab + (int64_t)r * 32, bar + st);
    }
  };
  issue(0, c0);
  issue(1, c0 + 1);
  for (int64_t c = c0; c < c1; c++) {
    const int st = (int)((c - c0) & 1), ph = (int)(((c - c0) >> 1) & 1);
    mbar_wait(bar + st, ph);
#pragma unroll 8
    for (int r = 0; r < ROWS; r++) {
      const float4 v = buf[((size_t)st * ROWS + r) * 32 + lane];
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    __syncwarp();
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    issue(st, c + 2);
  }
  if (acc.x + acc.y + acc.z + acc.w == 12345.f) out[0] = acc;
}

template <int ROWS, int WPB>
float run_tma(const float4 *tab, const int *idx, int64_t n, float4 *out, int blocks_per_sm, int sms) {
  const size_t smem = (size_t)WPB * 2 * ROWS * 512 + WPB * 16;
  CK(cudaFuncSetAttribute(replay_tma<ROWS, WPB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  replay_tma<ROWS, WPB><<<sms * blocks_per_sm, WPB * 32, smem>>>(tab, idx, n, out);
  CK(cudaGetLastError());
  CK(cudaEventRecord(a));
  const int it = 10;
  for (int i = 0; i < it; i++) replay_tma<ROWS, WPB><<<sms * blocks_per_sm, WPB * 32, smem>>>(tab, idx, n, out);
  CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return ms / it;
}

// LDGSTS variant: every lane cp.async-copies its 16 B of each row into a
// per-warp shared-memory ring (no registers held while in flight); rows are
// committed in groups of 4 and read back by the same lane (LDS.128), so in-
// flight depth is bounded by shared memory, not registers.  D rows in flight.
template <int D, int WPB, bool CG>
__global__ void __launch_bounds__(WPB * 32) replay_lds(const float4 *__restrict__ tab, const int *__restrict__ idx,
                                                        int64_t n_idx, float4 *__restrict__ out) {
  extern __shared__ __align__(128) float4 ring[];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  float4 *my = ring + (size_t)w * D * 32;
  const int64_t gw = (int64_t)blockIdx.x * WPB + w, nw = (int64_t)gridDim.x * WPB;
  const int64_t per = ((n_idx + nw - 1) / nw + 3) & ~int64_t(3);
  const int64_t q0 = gw * per, q1 = min(n_idx, q0 + per) & ~int64_t(3);
  float4 acc = make_float4(0, 0, 0, 0);
  constexpr int G = D / 4;  // groups of 4 rows in flight
  auto issue4 = [&](int64_t q) {  // rows q..q+3 into slots (q - q0) % D
    if (q < q1) {
#pragma unroll
      for (int u = 0; u < 4; u++) {
        const int r = __ldg(idx + q + u);
        const uint32_t d = (uint32_t)__cvta_generic_to_shared(my + (size_t)((q - q0 + u) % D) * 32 + lane);
        const float4 *src = tab + (int64_t)r * 32 + lane;
        if (CG) asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src) : "memory");
        else asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  for (int g = 0; g < G; g++) issue4(q0 + 4 * g);
  for (int64_t q = q0; q < q1; q += 4) {
    asm volatile("cp.async.wait_group %0;" ::"n"(G - 1) : "memory");
#pragma unroll
    for (int u = 0; u < 4; u++) {
      const float4 v = my[(size_t)((q - q0 + u) % D) * 32 + lane];
      acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
    }
    issue4(q + 4 * G);
  }
  asm volatile("cp.async.wait_all;" ::: "memory");
  if (acc.x + acc.y + acc.z + acc.w == 12345.f) out[0] = acc;
}

template <int D, int WPB, bool CG>
float run_lds(const float4 *tab, const int *idx, int64_t n, float4 *out, int bps, int sms) {
  const size_t smem = (size_t)WPB * D * 512;
  CK(cudaFuncSetAttribute(replay_lds<D, WPB, CG>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  replay_lds<D, WPB, CG><<<sms * bps, WPB * 32, smem>>>(tab, idx, n, out);
  CK(cudaGetLastError());
  CK(cudaEventRecord(a));
  const int it = 10;
  for (int i = 0; i < it; i++) replay_lds<D, WPB, CG><<<sms * bps, WPB * 32, smem>>>(tab, idx, n, out);
  CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return ms / it;
}

int main(int argc, char **argv) {
  if (argc < 4) { printf("usage: gather_replay cols.bin n_cols J\n"); return 1; }
  FILE *f = fopen(argv[1], "rb");
  if (!f) { printf("cannot open %s\n", argv[1]); return 1; }
  fseek(f, 0, SEEK_END); const int64_t n = ftell(f) / 4; fseek(f, 0, SEEK_SET);
  std::vector<int> h(n);
  if ((int64_t)fread(h.data(), 4, n, f) != n) { printf("short read\n"); return 1; }
  fclose(f);
  const int64_t K = atoll(argv[2]);
  const int J = atoi(argv[3]);
  if (J != 128) { printf("J must be 128\n"); return 1; }
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  int *idx; CK(cudaMalloc(&idx, n * 4));
  CK(cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice));
  float4 *tab; CK(cudaMalloc(&tab, K * J * 4));
  CK(cudaMemset(tab, 0, K * J * 4));
  float4 *out; CK(cudaMalloc(&out, 64));
  const double bytes = (double)n * J * 4;
  for (int occ : {2, 4, 8}) {
    const int blocks = sms * occ;
    float t4 = run<4, 0>(tab, idx, n, J / 4, out, blocks), t8 = run<8, 0>(tab, idx, n, J / 4, out, blocks),
          t16 = run<16, 0>(tab, idx, n, J / 4, out, blocks), t8n = run<8, 1>(tab, idx, n, J / 4, out, blocks);
    printf("{\"blocks_per_sm\": %d, \"ms_u4\": %.4f, \"ms_u8\": %.4f, \"ms_u16\": %.4f, \"ms_u8_nol1\": %.4f, "
           "\"gbs_u8\": %.0f, \"gathers\": %lld}\n", occ, t4, t8, t16, t8n, bytes / (t8 * 1e-3) / 1e9, (long long)n);
  }
  for (int occ : {2, 4, 8})
    printf("{\"interleaved_blocks_per_sm\": %d, \"ms_u4\": %.4f, \"ms_u8\": %.4f}\n", occ,
           run<4, 0, 1>(tab, idx, n, J / 4, out, sms * occ), run<8, 0, 1>(tab, idx, n, J / 4, out, sms * occ));
  if (getenv("LDS")) {
    printf("{\"lds_d8_w8_b4_cg\": %.4f, \"lds_d16_w8_b2_cg\": %.4f, \"lds_d16_w8_b3_cg\": %.4f, \"lds_d32_w8_b1_cg\": %.4f, "
           "\"lds_d16_w16_b1_cg\": %.4f, \"lds_d12_w8_b4_cg\": %.4f, \"lds_d16_w8_b3_ca\": %.4f, \"lds_d8_w16_b2_cg\": %.4f}\n",
           run_lds<8, 8, true>(tab, idx, n, out, 4, sms), run_lds<16, 8, true>(tab, idx, n, out, 2, sms),
           run_lds<16, 8, true>(tab, idx, n, out, 3, sms), run_lds<32, 8, true>(tab, idx, n, out, 1, sms),
           run_lds<16, 16, true>(tab, idx, n, out, 1, sms), run_lds<12, 8, true>(tab, idx, n, out, 4, sms),
           run_lds<16, 8, false>(tab, idx, n, out, 3, sms), run_lds<8, 16, true>(tab, idx, n, out, 2, sms));
  }
  if (getenv("NO_TMA")) return 0;
  printf("{\"tma_r16_w8_b1\": %.4f, \"tma_r32_w4_b1\": %.4f, \"tma_r32_w6_b1\": %.4f, \"tma_r16_w4_b2\": %.4f, \"tma_r8_w8_b2\": %.4f}\n",
         run_tma<16, 8>(tab, idx, n, out, 1, sms), run_tma<32, 4>(tab, idx, n, out, 1, sms),
         run_tma<32, 6>(tab, idx, n, out, 1, sms), run_tma<16, 4>(tab, idx, n, out, 2, sms),
         run_tma<8, 8>(tab, idx, n, out, 2, sms));
  return 0;
}
