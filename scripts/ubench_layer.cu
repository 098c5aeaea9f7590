// Micro-benchmark of the fixed per-layer costs of the interpreter loop on one
// CTA of 256 threads (B200): barrier, STS drain, ballot, dependent LDS.
// Build/run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ub scripts/ubench_layer.cu && /tmp/ub
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t lds(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

template <int V>
__global__ void k(unsigned long long* out, int iters, uint32_t seed) {
  __shared__ uint32_t S[4096];
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (uint32_t i = tid; i < 4096; i += 256) S[i] = (i * 7 + 1) & 1023;
  __syncthreads();
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(S);
  uint32_t x = seed + tid, acc = 0;
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; it++) {
    if (V >= 1) sts(base + 4 * (1024 + tid), x);
    if (V >= 2) {
      const uint32_t u = __ballot_sync(0xFFFFFFFFu, x & 1);
      if (lane == 0) sts(base + 4 * (2048 + warp), u ^ x);
    }
    if (V >= 3) x = lds(base + 4 * (x & 1023)) + 1;   // one dependent LDS
    if (V == 4 || V == 5) {                            // 32 independent LDS (gather-like)
      uint32_t a = 0;                                  // V4: conflict-free, V5: random banks
#pragma unroll
      for (int j = 0; j < 32; j++) {
        const uint32_t h = V == 4 ? (lane * 33u + j * 7u + (uint32_t)it) : ((lane * 2654435761u) ^ (j * 40503u) ^ (uint32_t)it * 977u) * 2246822519u >> 7;
        a |= __funnelshift_l(lds(base + 4 * (h & 1023)), 0, j) & (1u << j);
      }
      x ^= a;
    }
    if (V == 6) {                                      // fold5-like chain of 20 dependent LOP3s
#pragma unroll
      for (int j = 0; j < 20; j++) x = (x ^ (x >> 3)) & (x | 0x55u);
    }
    __syncthreads();
    acc += x;
  }
  unsigned long long t1 = clock64();
  if (tid == 0) out[0] = (t1 - t0) / iters;
  if (acc == 0x12345) out[1] = acc;
}

int main() {
  unsigned long long* d;
  cudaMalloc(&d, 16);
  unsigned long long h[2];
  const char* names[] = {"bar only", "+STS", "+ballot+STS", "+dep LDS", "+32 LDS no-conflict", "+32 LDS random", "+20 dep ALU (no LDS)"};
#define RUN(V)                                            \
  k<V><<<1, 256>>>(d, 100, 1);                            \
  k<V><<<1, 256>>>(d, 10000, 1);                          \
  cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);           \
  printf("%-18s %llu clocks/iter (1 CTA)\n", names[V], h[0]);
  RUN(0) RUN(1) RUN(2) RUN(3) RUN(4) RUN(5) RUN(6)
  return 0;
}
