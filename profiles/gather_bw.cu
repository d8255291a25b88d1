// Random row-gather bandwidth ceiling on this GPU (the memory pattern of phase S): every
// warp gathers rows of a row-major fp32 table [R × W] at uniformly random row ids, one
// 16-byte fragment per lane, U independent rows in flight per warp, and sums them (so the
// loads cannot be elided).  Reports gathered bytes / time for several table sizes (L2-
// resident up to ~100 MB; HBM beyond) and row widths (128 B = K 32, 512 B = K 128).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gather_bw profiles/gather_bw.cu
//   /tmp/gather_bw        (one JSON line per case)
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <vector>

template <int LPR, int U>  // lanes per row (W = 4·LPR floats), rows in flight per lane group
__global__ void __launch_bounds__(256) gather(const float4* __restrict__ tab, const int* __restrict__ idx,
                                              int64_t n, float* __restrict__ out) {
  constexpr int G = 32 / LPR;
  const int lane = threadIdx.x & 31, g = lane / LPR, lg = lane % LPR;
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int64_t base = warp * G * U; base < n; base += nwarps * G * U) {
    float4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u * G + g;
      const int r = i < n ? __ldg(idx + i) : 0;
      v[u] = __ldg(tab + (int64_t)r * LPR + lg);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      acc.x += v[u].x; acc.y += v[u].y; acc.z += v[u].z; acc.w += v[u].w;
    }
  }
  if (acc.x == 12345.f) out[0] = acc.y + acc.z + acc.w;
}

template <int LPR, int U>
float run(const float4* tab, const int* idx, int64_t n, float* out, int sms, int ctas_per_sm) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int grid = sms * ctas_per_sm;
  for (int i = 0; i < 3; ++i) gather<LPR, U><<<grid, 256>>>(tab, idx, n, out);
  cudaEventRecord(a);
  const int reps = 10;
  for (int i = 0; i < reps; ++i) gather<LPR, U><<<grid, 256>>>(tab, idx, n, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0.f;
  cudaEventElapsedTime(&ms, a, b);
  return ms / reps;
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int64_t n = 16 << 20;  // gathers per launch
  int* idx;
  float* out;
  cudaMalloc(&idx, n * sizeof(int));
  cudaMalloc(&out, 16);
  const int64_t max_bytes = 2048ll << 20;
  float4* tab;
  cudaMalloc(&tab, max_bytes);
  cudaMemset(tab, 0, max_bytes);
  std::vector<int> h(n);
  for (int W : {128, 32}) {
    const int row_bytes = W * 4;
    for (int64_t mb : {16, 32, 64, 96, 128, 256, 1024, 2048}) {
      const int64_t rows = (mb << 20) / row_bytes;
      uint64_t s = 88172645463325252ull;
      for (int64_t i = 0; i < n; ++i) {
        s ^= s << 13; s ^= s >> 7; s ^= s << 17;
        h[i] = (int)(s % (uint64_t)rows);
      }
      cudaMemcpy(idx, h.data(), n * sizeof(int), cudaMemcpyHostToDevice);
      for (int cps : {4, 8}) {
        float ms = W == 128 ? run<32, 4>(tab, idx, n, out, sms, cps) : run<8, 4>(tab, idx, n, out, sms, cps);
        const double gbs = (double)n * row_bytes / (ms * 1e-3) / 1e9;
        printf("{\"row_bytes\": %d, \"table_MB\": %lld, \"ctas_per_sm\": %d, \"ms\": %.4f, \"gather_GBs\": %.1f}\n",
               row_bytes, (long long)mb, cps, ms, gbs);
      }
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("{\"error\": \"%s\"}\n", cudaGetErrorString(e));
  return 0;
}
