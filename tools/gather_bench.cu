// tools/gather_bench.cu — B200 random-row-gather ceiling (measurement tool, not product).
//
// What the residual CSR SpMM does per stored entry is "fetch one row of the
// dense slice at a random index" (eq. 1; the SpMM of §III-A).
// This benchmark measures how many bytes per second the chip can deliver for
// exactly that access pattern, with nothing else in the kernel: a group of
// lanes fetches one row with 16-byte loads, U rows in flight per group, the
// rows summed into registers (so the loads are not dead).  Index streams are
// read coalesced with an evict-first hint like the SpMM's column stream.
//
//   rows of 64 / 128 / 176 / 256 / 512 B (w = 16, 32, 44, 64, 128 fp32)
//   table L2-resident (16-96 MB) or DRAM-resident (4 GB)
//   indices uniform, or power-law (i = floor(n * u^k): skew like R-MAT hubs)
//
// Output: one JSON line per case: delivered GB/s (row bytes / time, index
// bytes excluded and reported separately), best of 10 launches.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cmath>
#include <vector>
#include <algorithm>
#include <string>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

__device__ __forceinline__ int ld_cs(const int* p) {
  int v; asm volatile("ld.global.cs.b32 %0, [%1];" : "=r"(v) : "l"(p)); return v;
}
__device__ __forceinline__ float4 ld_nc(const float4* p) {
  float4 v;
  asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
  return v;
}

// G lanes per row, V float4 per lane (row = G*V float4), U rows in flight.
template <int G, int V, int U>
__global__ void __launch_bounds__(256) gather_kernel(const float4* __restrict__ tab, int ld4,
                                                     const int* __restrict__ idx, long long m,
                                                     float* __restrict__ sink) {
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const int sub = (int)(tid % G);
  const long long groups = (long long)gridDim.x * blockDim.x / G;
  const long long gid = tid / G;
  if (gid >= groups) return;
  float4 acc[V];
#pragma unroll
  for (int v = 0; v < V; ++v) acc[v] = make_float4(0.f, 0.f, 0.f, 0.f);
  for (long long base = gid * U; base < m; base += groups * U) {
    int r[U];
#pragma unroll
    for (int u = 0; u < U; ++u) r[u] = (base + u < m) ? ld_cs(idx + base + u) : -1;
    float4 x[U][V];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v)
        x[u][v] = r[u] >= 0 ? ld_nc(tab + (long long)r[u] * ld4 + sub + v * G)
                            : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < V; ++v) {
        acc[v].x += x[u][v].x; acc[v].y += x[u][v].y; acc[v].z += x[u][v].z; acc[v].w += x[u][v].w;
      }
  }
  float s = 0.f;
#pragma unroll
  for (int v = 0; v < V; ++v) s += acc[v].x + acc[v].y + acc[v].z + acc[v].w;
  if (s == 12345.678f) sink[0] = s;   // keeps the loads live
}

static uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

struct Case { const char* name; int row_floats; };

template <int G, int V, int U>
static float run(const float4* tab, int ld4, const int* idx, long long m, float* sink, int grid) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  for (int i = 0; i < 3; ++i) gather_kernel<G, V, U><<<grid, 256>>>(tab, ld4, idx, m, sink);
  CK(cudaGetLastError());
  float best = 1e30f;
  for (int i = 0; i < 10; ++i) {
    CK(cudaEventRecord(a));
    gather_kernel<G, V, U><<<grid, 256>>>(tab, ld4, idx, m, sink);
    CK(cudaEventRecord(b));
    CK(cudaEventSynchronize(b));
    float ms; CK(cudaEventElapsedTime(&ms, a, b));
    best = std::min(best, ms);
  }
  CK(cudaEventDestroy(a)); CK(cudaEventDestroy(b));
  return best;
}

int main(int argc, char** argv) {
  int dev = 0; CK(cudaSetDevice(dev));
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  const int sms = p.multiProcessorCount;
  int clk = 0; CK(cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev));
  fprintf(stderr, "device %s, %d SMs, L2 %d MB\n", p.name, sms, p.l2CacheSize >> 20);
  const long long m = 64ll << 20;               // 64 M gathered rows per launch
  std::vector<int> h(m);
  int* idx; CK(cudaMalloc(&idx, m * sizeof(int)));
  float* sink; CK(cudaMalloc(&sink, 4));
  const size_t big = 4ull << 30;                 // 4 GB DRAM-resident table
  float4* tab; CK(cudaMalloc(&tab, big));
  CK(cudaMemset(tab, 0, big));
  const int row_floats[] = {16, 32, 44, 64, 128};
  const double tables_mb[] = {16, 48, 96, 4096};
  for (int rf : row_floats) {
    const int ld4 = rf / 4;
    const double row_b = rf * 4.0;
    for (double tmb : tables_mb) {
      const long long n = (long long)(tmb * 1048576.0 / row_b);
      for (int dist = 0; dist < 2; ++dist) {
        for (long long i = 0; i < m; ++i) {
          const double u = (sm64(i * 2 + dist * 0x5555 + rf * 7919) >> 11) * (1.0 / 9007199254740992.0);
          long long r = dist == 0 ? (long long)(u * n) : (long long)(n * std::pow(u, 4.0));
          if (r >= n) r = n - 1;
          // power-law: spread the hot low indices over the table (like a permuted graph)
          if (dist == 1) r = (long long)((sm64((uint64_t)r) % (uint64_t)n));
          h[i] = (int)r;
        }
        CK(cudaMemcpy(idx, h.data(), m * sizeof(int), cudaMemcpyHostToDevice));
        const int grid = sms * 8;
        float ms = 0;
        switch (rf) {
          case 16: ms = run<4, 1, 4>(tab, ld4, idx, m, sink, grid); break;
          case 32: ms = run<8, 1, 4>(tab, ld4, idx, m, sink, grid); break;
          case 44: ms = run<11, 1, 4>(tab, ld4, idx, m, sink, grid); break;
          case 64: ms = run<16, 1, 4>(tab, ld4, idx, m, sink, grid); break;
          case 128: ms = run<32, 1, 4>(tab, ld4, idx, m, sink, grid); break;
        }
        float ms2 = 0;   // the fp32 SpMM's own lane mapping for 512 B rows (G = 8, V = 4)
        if (rf == 128) ms2 = run<8, 4, 1>(tab, ld4, idx, m, sink, grid);
        const double gbs = m * row_b / (ms * 1e-3) / 1e9;
        printf("{\"row_bytes\": %d, \"table_mb\": %.0f, \"dist\": \"%s\", \"rows\": %lld, "
               "\"ms\": %.4f, \"delivered_gbs\": %.1f, \"bytes_per_clk\": %.1f, \"index_gbs\": %.1f, "
               "\"spmm_mapping_g8v4_gbs\": %.1f}\n",
               (int)row_b, tmb, dist ? "powerlaw" : "uniform", m, ms, gbs,
               gbs * 1e9 / (clk * 1e3), m * 4.0 / (ms * 1e-3) / 1e9,
               ms2 > 0 ? m * row_b / (ms2 * 1e-3) / 1e9 : 0.0);
        fflush(stdout);
      }
    }
  }
  return 0;
}
