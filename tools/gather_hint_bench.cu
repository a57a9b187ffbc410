// tools/gather_hint_bench.cu — does an L2 eviction-priority hint on the
// gathered rows raise the L2 hit rate of a skewed (power-law) gather over a
// table much larger than L2?  (measurement tool, not product)
//
// Index stream: rank r = floor(n * u^k) (hot ranks first), spread over the
// table by a hash (a permuted graph).  The hint bit (bit 31 of the index) is
// set when r >= H ("cold").  Variants:
//   plain : ld.global.nc for every row
//   hint  : cold rows ld.global.nc.L2::cache_hint with an evict_first policy,
//           hot rows with an evict_last policy (per-lane policy operand, no
//           divergence)
//   first : cold rows evict_first, hot rows default policy
// Rows of 1 KB (w = 256 fp32) and 512 B, table 2.5 GB (2.45 M rows: the
// products-shaped column slice at P = 1).
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cmath>
#include <vector>
#include <algorithm>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ int ld_cs(const int* p) {
  int v; asm volatile("ld.global.cs.b32 %0, [%1];" : "=r"(v) : "l"(p)); return v;
}
__device__ __forceinline__ float4 ld_pol(const float4* p, uint64_t pol) {
  float4 v;
  asm volatile("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
  return v;
}
__device__ __forceinline__ float4 ld_nc(const float4* p) {
  float4 v;
  asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}

// MODE 0 plain, 1 hint (cold first / hot last), 2 cold first only
template <int G, int V, int MODE>
__global__ void __launch_bounds__(256) gather_kernel(const float4* __restrict__ tab, int ld4,
                                                     const int* __restrict__ idx, long long m,
                                                     float* __restrict__ sink) {
  uint64_t pol_first, pol_last, pol_norm;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol_first));
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_last));
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol_norm));
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const int sub = (int)(tid % G);
  const long long groups = (long long)gridDim.x * blockDim.x / G;
  const long long gid = tid / G;
  if (gid >= groups) return;
  constexpr int U = 4;
  float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
  for (long long base = gid * U; base < m; base += groups * U) {
    int r[U];
#pragma unroll
    for (int u = 0; u < U; ++u) r[u] = (base + u < m) ? ld_cs(idx + base + u) : -1;
    float4 x[U][V];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const bool cold = r[u] < 0 && r[u] != -1;
      const int row = r[u] & 0x7fffffff;
      const uint64_t pol = cold ? pol_first : (MODE == 1 ? pol_last : pol_norm);
#pragma unroll
      for (int v = 0; v < V; ++v) {
        const float4* p = tab + (long long)row * ld4 + sub + v * G;
        if (r[u] == -1) x[u][v] = make_float4(0.f, 0.f, 0.f, 0.f);
        else x[u][v] = MODE == 0 ? ld_nc(p) : ld_pol(p, pol);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v) {
        acc.x += x[u][v].x; acc.y += x[u][v].y; acc.z += x[u][v].z; acc.w += x[u][v].w;
      }
  }
  const float s = acc.x + acc.y + acc.z + acc.w;
  if (s == 12345.678f) sink[0] = s;
}

static uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

template <int G, int V, int MODE>
static float run(const float4* tab, int ld4, const int* idx, long long m, float* sink, int grid) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  gather_kernel<G, V, MODE><<<grid, 256>>>(tab, ld4, idx, m, sink);
  CK(cudaGetLastError());
  float best = 1e30f;
  for (int i = 0; i < 5; ++i) {
    CK(cudaEventRecord(a));
    gather_kernel<G, V, MODE><<<grid, 256>>>(tab, ld4, idx, m, sink);
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b));
    best = std::min(best, ms);
  }
  return best;
}

int main() {
  CK(cudaSetDevice(0));
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  const int grid = p.multiProcessorCount * 8;
  const long long n = 2449029;
  const long long m = 32ll << 20;
  std::vector<int> h(m);
  int* idx; CK(cudaMalloc(&idx, m * sizeof(int)));
  float* sink; CK(cudaMalloc(&sink, 4));
  float4* tab; CK(cudaMalloc(&tab, (size_t)n * 1024));
  CK(cudaMemset(tab, 0, (size_t)n * 1024));
  for (double k : {6.0, 9.0}) {
    for (long long H : {0ll, 40000ll, 80000ll, 120000ll, 200000ll}) {
      for (long long i = 0; i < m; ++i) {
        const double u = (sm64(i * 7 + (long long)k) >> 11) * (1.0 / 9007199254740992.0);
        long long r = (long long)(n * std::pow(u, k));
        if (r >= n) r = n - 1;
        int row = (int)(sm64((uint64_t)r + 99) % (uint64_t)n);
        h[i] = row | ((H > 0 && r >= H) ? (int)0x80000000u : 0);
      }
      CK(cudaMemcpy(idx, h.data(), m * sizeof(int), cudaMemcpyHostToDevice));
      for (int rb : {1024, 512}) {
        const int ld4 = 64;   // table rows always 1 KB apart (the slice's leading dim)
        float t0, t1, t2;
        if (rb == 1024) {
          t0 = run<32, 2, 0>(tab, ld4, idx, m, sink, grid);
          t1 = run<32, 2, 1>(tab, ld4, idx, m, sink, grid);
          t2 = run<32, 2, 2>(tab, ld4, idx, m, sink, grid);
        } else {
          t0 = run<32, 1, 0>(tab, ld4, idx, m, sink, grid);
          t1 = run<32, 1, 1>(tab, ld4, idx, m, sink, grid);
          t2 = run<32, 1, 2>(tab, ld4, idx, m, sink, grid);
        }
        auto gbs = [&](float ms) { return m * (double)rb / (ms * 1e-3) / 1e9; };
        printf("{\"k\": %.0f, \"hot_rows\": %lld, \"row_bytes\": %d, \"plain_gbs\": %.0f, \"hint_gbs\": %.0f, "
               "\"cold_first_gbs\": %.0f}\n", k, H, rb, gbs(t0), gbs(t1), gbs(t2));
        fflush(stdout);
      }
    }
  }
  return 0;
}
