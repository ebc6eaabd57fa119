// Philox4x32-10 throughput probe: the ALU roof of the IC sampler on this GPU.
// Every thread runs ITER iterations of ILP independent Philox chains on
// distinct counters and folds the words into one value (kept live).
// Reports Philox calls/s and words/s (= examined-edge draws/s).
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_sc_doneyhl25_b200/csrc/philox.cuh"

using namespace eim;

template <int ILP>
__global__ void __launch_bounds__(256) roof(uint64_t seed, uint32_t iters, uint32_t* out) {
  const PhiloxKey K = philox_key(seed);
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t acc = 0;
  for (uint32_t it = 0; it < iters; ++it) {
    uint4 w[ILP];
#pragma unroll
    for (int k = 0; k < ILP; ++k) w[k] = philox_at(((uint64_t)it * ILP + k) << 20 | tid, 12345, TAG_EDGE, K);
#pragma unroll
    for (int k = 0; k < ILP; ++k) acc ^= min(min(w[k].x, w[k].y), min(w[k].z, w[k].w));
  }
  if (acc == 0x12345678u) out[tid] = acc;
}

// The sampler's form: one sample per thread, quads varying (philox_edge: the
// sample-constant work of rounds 0-1 hoisted, 18 wide multiplies per call).
template <int ILP>
__global__ void __launch_bounds__(256) roof_edge(uint64_t seed, uint32_t iters, uint32_t* out) {
  const PhiloxKey K = philox_key(seed);
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const EdgeConsts E = edge_consts(0u, (uint32_t)(tid * 2654435761u), ctr_hi(tid, TAG_EDGE), K);
  uint32_t acc = 0;
  for (uint32_t it = 0; it < iters; ++it) {
    uint4 w[ILP];
#pragma unroll
    for (int k = 0; k < ILP; ++k) w[k] = philox_edge((uint32_t)(it * ILP + k), E, K);
#pragma unroll
    for (int k = 0; k < ILP; ++k) acc ^= min(min(w[k].x, w[k].y), min(w[k].z, w[k].w));
  }
  if (acc == 0x12345678u) out[tid] = acc;
}

template <int ILP>
void run_edge(int sms) {
  uint32_t* out;
  cudaMalloc(&out, 1 << 24);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int blocks_per_sm : {4, 8}) {
    const uint32_t blocks = sms * blocks_per_sm, iters = 4096 / ILP;
    roof_edge<ILP><<<blocks, 256>>>(1, 16, out);
    cudaEventRecord(a);
    roof_edge<ILP><<<blocks, 256>>>(1, iters, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double calls = (double)blocks * 256 * iters * ILP;
    printf("{\"form\": \"philox_edge\", \"ilp\": %d, \"blocks_per_sm\": %d, \"ms\": %.3f, \"philox_per_s\": %.4e, "
           "\"words_per_s\": %.4e}\n", ILP, blocks_per_sm, ms, calls / ms * 1e3, 4 * calls / ms * 1e3);
  }
  cudaFree(out);
}

template <int ILP>
void run(int sms) {
  uint32_t* out;
  cudaMalloc(&out, 1 << 24);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  for (int blocks_per_sm : {4, 8}) {
    const uint32_t blocks = sms * blocks_per_sm, iters = 4096 / ILP;
    roof<ILP><<<blocks, 256>>>(1, 16, out);
    cudaEventRecord(a);
    roof<ILP><<<blocks, 256>>>(1, iters, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double calls = (double)blocks * 256 * iters * ILP;
    printf("{\"ilp\": %d, \"blocks_per_sm\": %d, \"ms\": %.3f, \"philox_per_s\": %.4e, \"words_per_s\": %.4e}\n",
           ILP, blocks_per_sm, ms, calls / ms * 1e3, 4 * calls / ms * 1e3);
  }
  cudaFree(out);
}

// One 256-thread group alone on the GPU (the latency-bound case of a heavy
// sampler batch): ns per iteration of ILP chains per thread.
template <int ILP>
void single() {
  uint32_t* out;
  cudaMalloc(&out, 1 << 20);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const uint32_t iters = 4096;
  roof<ILP><<<1, 256>>>(1, 16, out);
  cudaEventRecord(a);
  roof<ILP><<<1, 256>>>(1, iters, out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  printf("{\"single_group_ilp\": %d, \"ns_per_iter\": %.1f, \"quads_per_ns\": %.3f}\n", ILP, ms * 1e6 / iters,
         256.0 * ILP * iters / (ms * 1e6));
  cudaFree(out);
}

int main(int argc, char** argv) {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  if (argc > 1) {  // latency probe
    single<1>();
    single<2>();
    single<4>();
    return 0;
  }
  run<1>(sms);
  run<2>(sms);
  run<4>(sms);
  run_edge<1>(sms);
  run_edge<2>(sms);
  run_edge<4>(sms);
  return 0;
}
