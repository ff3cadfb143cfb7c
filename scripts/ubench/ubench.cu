// Throughput microbenchmarks of the shared-memory / warp primitives the graph kernels use
// (cycles per warp-instruction per SM, all SMs busy).  nvcc -arch=sm_100a -O3 ubench.cu
#include <cstdio>
#include <cuda_runtime.h>

constexpr int ITERS = 4096;

template <int OP>
__global__ void k(int* out, int seed) {
  __shared__ int s[8192];
  for (int i = threadIdx.x; i < 8192; i += blockDim.x) s[i] = i;
  __syncthreads();
  int acc = seed + threadIdx.x;
  unsigned addr = (threadIdx.x * 33u + blockIdx.x) & 8191u;  // spread over banks
  long long t0 = clock64();
#pragma unroll 4
  for (int it = 0; it < ITERS; ++it) {
    if (OP == 0) acc += atomicAdd(&s[addr], 1);                   // ATOMS.ADD spread
    if (OP == 1) acc += atomicCAS(&s[addr], acc, acc + 1);         // ATOMS.CAS spread
    if (OP == 2) { atomicAdd(&s[addr], 1); }                       // RED.ADD (no return)
    if (OP == 3) acc += __match_any_sync(0xffffffffu, acc & 7);    // MATCH.ANY
    if (OP == 4) acc += __shfl_sync(0xffffffffu, acc, (threadIdx.x + it) & 31);  // SHFL
    if (OP == 5) acc += s[(addr + it * 32) & 8191];                // LDS spread, conflict-free
    if (OP == 6) { s[(addr + it * 32) & 8191] = acc; acc += 1; }   // STS
    if (OP == 7) { atomicOr((unsigned*)&s[addr], 1u << (it & 31)); } // ATOMS.OR no return
    if (OP == 8) acc += __reduce_add_sync(0xffffffffu, acc);       // REDUX
    if (OP == 9) acc += __popc(__ballot_sync(0xffffffffu, acc & 1)); // VOTE+POPC
    if (OP == 10) { float* f = (float*)s; atomicAdd(&f[addr], 1.0f); }  // float smem add (CAS loop?)
    if (OP == 11) acc += atomicAdd(&s[(it & 7) * 1024 + (threadIdx.x & 31)], 1);  // ATOMS, 32 distinct banks
    addr = (addr + 97u) & 8191u;
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x] = (int)((t1 - t0));
  if (acc == 123456789) out[0] = acc;
}

template <int OP>
void run(const char* name, int threads, int blocks_per_sm) {
  int* d;
  cudaMalloc(&d, 148 * 64 * sizeof(int));
  int grid = 148 * blocks_per_sm;
  k<OP><<<grid, threads>>>(d, 1);
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a);
  k<OP><<<grid, threads>>>(d, 2);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  double warp_instr_per_sm = (double)threads / 32 * blocks_per_sm * ITERS;
  double cyc = ms * 1e-3 * 1.9e9;  // approx SM clock
  printf("%-28s threads/SM %5d: %.3f ms  -> %.2f cycles per warp-instr per SM, %.3f lanes/cycle\n", name,
         threads * blocks_per_sm, ms, cyc / warp_instr_per_sm, warp_instr_per_sm * 32 / cyc);
  cudaFree(d);
}

int main() {
  for (int bps : {4, 8}) {
    run<0>("ATOMS.ADD (return)", 256, bps);
    run<1>("ATOMS.CAS", 256, bps);
    run<2>("ATOMS.ADD (no return)", 256, bps);
    run<7>("ATOMS.OR (no return)", 256, bps);
    run<10>("smem float atomicAdd", 256, bps);
    run<11>("ATOMS.ADD 32 banks", 256, bps);
    run<3>("MATCH.ANY", 256, bps);
    run<4>("SHFL", 256, bps);
    run<5>("LDS", 256, bps);
    run<6>("STS", 256, bps);
    run<8>("REDUX.ADD", 256, bps);
    run<9>("VOTE.BALLOT+POPC", 256, bps);
  }
  return 0;
}
