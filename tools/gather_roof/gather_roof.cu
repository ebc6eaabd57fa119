// Random dependent-load probe: the roof of the LT walk kernel (one random
// 16-B walk-store entry per step, the next address taken from the entry,
// plus one membership-table CAS per step).  W walkers (threads) each follow
// a chain of S dependent random 16-B loads over a buffer of the walk store's
// size (C3: 117,185,083 entries = 1.9 GB); with --cas every step also CASes a
// random 8-B slot of a table of the C3 round's size (2^25 slots).  Reports
// steps/s for the C3 round's concurrency (58,277 walkers) and for a full GPU
// (2048 threads per SM).
#include <cstdio>
#include <cstdint>
#include <cstring>

__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 33;
  x *= 0xff51afd7ed558ccdull;
  x ^= x >> 33;
  x *= 0xc4ceb9fe1a85ec53ull;
  x ^= x >> 33;
  return x;
}

__global__ void fill(uint4* buf, uint64_t n) {
  for (uint64_t e = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n; e += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t nx = mix(e * 0x9E3779B97F4A7C15ull + 1) % n;
    buf[e] = make_uint4((uint32_t)nx, (uint32_t)(nx >> 32), (uint32_t)e, 0u);
  }
}

__global__ void __launch_bounds__(256) chase(const uint4* __restrict__ buf, uint64_t n, unsigned long long* table,
                                             uint32_t tbits, uint32_t walkers, uint32_t steps, uint32_t* out) {
  const uint32_t w = blockIdx.x * blockDim.x + threadIdx.x;
  if (w >= walkers) return;
  uint64_t idx = mix(w + 12345ull) % n;
  uint32_t acc = 0;
  for (uint32_t s = 0; s < steps; ++s) {
    const uint4 e = __ldg(buf + idx);
    if (table) {
      const uint64_t h = mix(((uint64_t)w << 32) | e.z) >> (64 - tbits);
      acc += (uint32_t)atomicCAS(table + h, 0ull, ((uint64_t)(w + 1) << 32) | e.z);
    }
    idx = ((uint64_t)e.y << 32 | e.x);
    acc += e.z;
  }
  if (acc == 0x12345678u) out[w] = acc;
}

int main(int argc, char** argv) {
  const bool cas = argc > 1 && !strcmp(argv[1], "--cas");
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const uint64_t n = 117185083ull;
  const uint32_t tbits = 25;
  uint4* buf;
  unsigned long long* table = nullptr;
  uint32_t* out;
  if (cudaMalloc(&buf, n * sizeof(uint4)) != cudaSuccess) return 1;
  cudaMalloc(&out, 4u << 20);
  if (cas) cudaMalloc(&table, (8ull << tbits));
  fill<<<sms * 8, 256>>>(buf, n);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const uint32_t walkers_list[2] = {58277u, (uint32_t)sms * 2048u};
  for (uint32_t walkers : walkers_list) {
    const uint32_t steps = 256;
    for (int rep = 0; rep < 2; ++rep) {
      if (table) cudaMemset(table, 0, 8ull << tbits);
      cudaEventRecord(a);
      chase<<<(walkers + 255) / 256, 256>>>(buf, n, table, tbits, walkers, steps, out);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (rep == 1)
        printf("{\"probe\": \"random 16-B dependent loads%s\", \"walkers\": %u, \"steps\": %u, \"ms\": %.3f, "
               "\"steps_per_s\": %.4e, \"us_per_step\": %.3f}\n",
               cas ? " + table CAS" : "", walkers, steps, ms, (double)walkers * steps / ms * 1e3, ms * 1e3 / steps);
    }
  }
  return 0;
}
