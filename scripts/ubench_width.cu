// Micro-benchmark: a dense boomerang layer (8192 leaves, random state words,
// records from shared memory, levels up to 10, write-outs, block barrier) as
// (A) 256 threads x 32 leaves (the current ISA: fold5 in-thread, ballot, fold5)
// (B) 512 threads x 16 leaves (fold4 in-thread, ballot, fold5 over the warp).
// One CTA per SM; clocks per layer on CTA 0.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/uw scripts/ubench_width.cu && /tmp/uw
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t bsel(uint32_t a, uint32_t b, uint32_t m) { return (a & ~m) | (b & m); }
__device__ __forceinline__ uint32_t fold5(uint32_t v, uint32_t xa, uint32_t xb, uint32_t ob) {
  const uint32_t r1 = (v ^ xa) & (((v >> 16) ^ xb) | ob);
  const uint32_t r2 = ((r1 << 16) ^ xa) & (((r1 << 8) ^ xb) | ob);
  const uint32_t r3 = ((r2 << 8) ^ xa) & (((r2 << 4) ^ xb) | ob);
  const uint32_t r4 = ((r3 << 4) ^ xa) & (((r3 << 2) ^ xb) | ob);
  const uint32_t r5 = ((r4 << 2) ^ xa) & (((r4 << 1) ^ xb) | ob);
  return bsel(bsel(bsel(bsel(r1, r2, 0x00FF0000u), r3, 0x0F000000u), r4, 0x30000000u), r5, 0xC0000000u) & 0x7FFFFFFFu;
}
// levels 1-4 of 16 leaves in bits [0,16): L1 [0,8) A=v[q] B=v[q+8]; L2 [8,12); L3 [12,14); L4 [14]
__device__ __forceinline__ uint32_t fold4(uint32_t v, uint32_t xa, uint32_t xb, uint32_t ob) {
  const uint32_t r1 = (v ^ xa) & (((v >> 8) ^ xb) | ob);
  const uint32_t r2 = ((r1 << 8) ^ xa) & (((r1 << 4) ^ xb) | ob);
  const uint32_t r3 = ((r2 << 4) ^ xa) & (((r2 << 2) ^ xb) | ob);
  const uint32_t r4 = ((r3 << 2) ^ xa) & (((r3 << 1) ^ xb) | ob);
  return bsel(bsel(bsel(r1, r2, 0x0F00u), r3, 0x3000u), r4, 0x4000u) & 0x7FFFu;
}

template <int T, int NL>   // threads, leaves per thread
__global__ void __launch_bounds__(T, 1) lk(unsigned long long* out, int iters) {
  extern __shared__ __align__(16) uint32_t sm[];
  constexpr int NQ = NL / 8;                       // uint4 of u16 entries per lane
  constexpr int NLAY = 4;
  constexpr int WREC = 4 + 128 + 128 * NQ;         // per warp
  constexpr int NW = T / 32;
  uint32_t* S = sm;                                // 2048 words
  uint32_t* area = sm + 2048;
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (uint32_t i = tid; i < 2048; i += T) S[i] = i * 2654435761u;
  for (uint32_t i = tid; i < NLAY * NW * WREC; i += T) {
    const uint32_t h = i * 2246822519u + 12345u;
    // two u16 entries: rot | word << 5 (word < 2048)
    area[i] = ((h & 31u) | (((h >> 5) & 2047u) << 5)) | ((((h >> 16) & 31u) | (((h >> 21) & 2047u) << 5)) << 16);
  }
  __syncthreads();
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(S);
  uint32_t acc = 0;
  unsigned long long t0 = 0;
  for (int it = 0; it < iters; it++) {
    if (it == 16) t0 = clock64();
    const uint32_t* rec = area + ((it % NLAY) * NW + warp) * WREC;
    const uint4 wc = *reinterpret_cast<const uint4*>(rec);
    const uint4 lc = *(reinterpret_cast<const uint4*>(rec + 4) + lane);
    uint4 e[NQ];
#pragma unroll
    for (int g = 0; g < NQ; g++) e[g] = *(reinterpret_cast<const uint4*>(rec + 4 + 128 + 128 * g) + lane);
    uint32_t accv[4] = {0, 0, 0, 0};
#pragma unroll
    for (int g = 0; g < NQ; g++) {
      const uint32_t q[4] = {e[g].x, e[g].y, e[g].z, e[g].w};
#pragma unroll
      for (int k = 0; k < 4; k++) {
        uint32_t lo, hi;
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(lo) : "r"(sb + ((q[k] >> 3) & 0x1FFCu)));
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(hi) : "r"(sb + ((q[k] >> 19) & 0x1FFCu)));
        accv[k] |= (__funnelshift_l(lo, lo, q[k]) & (1u << (8 * g + 2 * k))) |
                   (__funnelshift_l(hi, hi, q[k] >> 16) & (1u << (8 * g + 2 * k + 1)));
      }
    }
    const uint32_t v = (accv[0] | accv[1]) | (accv[2] | accv[3]);
    uint32_t P, top;
    if (NL == 32) { P = fold5(v, lc.x, lc.y, lc.z); top = (P >> 30) & 1u; }
    else { P = fold4(v, lc.x, lc.y, lc.z); top = (P >> 14) & 1u; }
    if (lc.w & 1) asm volatile("st.shared.u32 [%0], %1;" ::"r"(sb + 4 * (1024 + (tid & 511))), "r"(P) : "memory");
    const uint32_t u = __ballot_sync(0xFFFFFFFFu, top);
    const uint32_t Pw = fold5(u, wc.x, wc.y, wc.z);
    if (lane == 0 && (wc.w & 1)) asm volatile("st.shared.u32 [%0], %1;" ::"r"(sb + 4 * (1600 + warp)), "r"(Pw) : "memory");
    acc += P ^ Pw;
    __syncthreads();
  }
  unsigned long long t1 = clock64();
  if (tid == 0 && blockIdx.x == 0) out[0] = (t1 - t0) / (iters - 16);
  if (acc == 0x12345u) out[1] = acc;
}

template <int T, int NL>
void run(const char* name, unsigned long long* d, int sms) {
  constexpr int NQ = NL / 8, NW = T / 32, WREC = 4 + 128 + 128 * NQ;
  const int smem = (2048 + 4 * NW * WREC) * 4 + 16;
  cudaFuncSetAttribute(lk<T, NL>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  lk<T, NL><<<sms, T, smem>>>(d, 100);
  lk<T, NL><<<sms, T, smem>>>(d, 2016);
  cudaDeviceSynchronize();
  unsigned long long h = 0;
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("%-50s %6llu clk/layer (%s)\n", name, h, cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long* d;
  cudaMalloc(&d, 16);
  run<256, 32>("A: 256 threads x 32 leaves (current)", d, sms);
  run<512, 16>("B: 512 threads x 16 leaves", d, sms);
  run<256, 16>("C: 256 threads x 16 leaves (half layer, ref)", d, sms);
  return 0;
}
