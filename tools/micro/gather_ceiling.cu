// Random-row gather ceiling on one B200 (tools/micro; not part of the library).
// Table: n rows x 208 B (products' bf16 feature store: 100 columns padded to 104).
// Reads R row ids (16 lanes per row, 13 x 16 B each, UNROLL rows in flight per lane
// group), XOR-folds each row to one word so nothing is dead.  Three id streams:
//   uniq_sorted  : the U unique sources in ascending id order (what a source-major pass reads)
//   uniq_random  : the same U rows in random order
//   edges        : E ids with duplicates (each unique row drawn ~E/U times, random order),
//                  the layer-1 gather's access stream
// Prints GB/s of row bytes actually read (R x 208) and of unique bytes (U x 208).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <algorithm>
#include <cstdlib>
#include <cuda_runtime.h>

template <int UNROLL>
__global__ void __launch_bounds__(256) gather(const uint4* __restrict__ tab, int pitch16, const int* __restrict__ ids,
                                              int n_ids, uint32_t* out) {
  const int l = threadIdx.x & 15;
  const int lv = l < 13 ? l : 0;
  const int groups = gridDim.x * (blockDim.x >> 4);
  int g = (blockIdx.x * blockDim.x + threadIdx.x) >> 4;
  for (int base = g * UNROLL; base < n_ids; base += groups * UNROLL) {
    uint4 v[UNROLL];
#pragma unroll
    for (int q = 0; q < UNROLL; ++q) {
      const int i = base + q;
      const int u = i < n_ids ? __ldg(ids + i) : 0;
      v[q] = __ldg(tab + int64_t(u) * pitch16 + lv);
    }
    uint32_t x = 0;
#pragma unroll
    for (int q = 0; q < UNROLL; ++q) x ^= v[q].x ^ v[q].y ^ v[q].z ^ v[q].w;
    if (x == 0x12345678u) out[g] = x;
  }
}

int main(int argc, char** argv) {
  // scale 1: products' layer-1 block; scale 10: the same density over a 10x table (amortises
  // the ~2-4 us of launch latency the events include)
  const int64_t sc = argc > 1 ? atoi(argv[1]) : 1;
  const int64_t n = 2400000 * sc, pitch = 208, U = 217337 * sc, E = 482282 * sc;
  uint4* tab; cudaMalloc(&tab, n * pitch); cudaMemset(tab, 1, n * pitch);
  uint32_t* out; cudaMalloc(&out, 1 << 24);
  char* flush; const size_t fl = size_t(256) << 20; cudaMalloc(&flush, fl);
  std::mt19937_64 rng(7);
  std::vector<int> all(n); for (int64_t i = 0; i < n; ++i) all[i] = int(i);
  std::shuffle(all.begin(), all.end(), rng);
  std::vector<int> uniq(all.begin(), all.begin() + U);
  std::vector<int> srt = uniq; std::sort(srt.begin(), srt.end());
  std::vector<int> edges(E);
  for (int64_t e = 0; e < E; ++e) edges[e] = uniq[e < U ? e : rng() % U];
  std::shuffle(edges.begin(), edges.end(), rng);
  struct S { const char* name; std::vector<int>* v; } streams[] = {{"uniq_sorted", &srt}, {"uniq_random", &uniq}, {"edges", &edges}};
  int* d_ids; cudaMalloc(&d_ids, E * 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  for (auto& s : streams) {
    cudaMemcpy(d_ids, s.v->data(), s.v->size() * 4, cudaMemcpyHostToDevice);
    for (int bpsm : {4, 8}) {
      for (int unroll : {4, 8, 16}) {
        float best = 1e9;
        for (int rep = 0; rep < 5; ++rep) {
          cudaMemset(flush, rep, fl);
          cudaEventRecord(a);
          const int nid = int(s.v->size());
          if (unroll == 4) gather<4><<<sms * bpsm, 256>>>(tab, pitch / 16, d_ids, nid, out);
          else if (unroll == 8) gather<8><<<sms * bpsm, 256>>>(tab, pitch / 16, d_ids, nid, out);
          else gather<16><<<sms * bpsm, 256>>>(tab, pitch / 16, d_ids, nid, out);
          cudaEventRecord(b); cudaEventSynchronize(b);
          float ms; cudaEventElapsedTime(&ms, a, b); best = std::min(best, ms);
        }
        const double rows = double(s.v->size());
        printf("x%lld %-12s bpsm %d unroll %2d: %7.2f us  %7.0f GB/s of rows read  %7.0f GB/s of unique rows\n", (long long)sc, s.name, bpsm,
               unroll, best * 1e3, rows * pitch / (best * 1e-3) / 1e9, double(U) * pitch / (best * 1e-3) / 1e9);
      }
    }
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
