// Micro-benchmark of a *light* interpreter layer (few leaves per thread), built
// up step by step to price each per-layer cost of gem_step_kernel's loop:
//   V0 sparse gather (4 leaves/thread) + fold5 + ballot + fold5 + write-out STS + __syncthreads
//   V1 + next layer's records loaded from shared memory (header, warp consts, lane consts, 1 leaf group)
//   V2 + levels 11-13 hand-off (bar.arrive by warps 1-7, warp 0 bar.sync + fold3 + STS)
//   V3 + one mbarrier try_wait (already complete) per layer by every thread
//   V4 = V2 with the records loaded two layers ahead (double-buffered registers)
// One CTA of 256 threads per SM, grid = #SMs; clocks per layer on CTA 0.
// Build/run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ul scripts/ubench_layer2.cu && /tmp/ul
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
struct Regs { uint4 e, e2[4], lc, wc, hd; };
constexpr int NLAY = 4;
constexpr int REC_WORDS = 4 + 128 + 128 * 5;   // per warp: wc, lane consts, 5 leaf groups
__device__ __forceinline__ void load_rec(const uint32_t* area, int l, Regs& R) {
  const uint32_t lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const uint32_t* L = area + l * (16 + 8 * REC_WORDS);
  R.hd = *reinterpret_cast<const uint4*>(L);
  const uint32_t* rec = L + 16 + warp * REC_WORDS;
  R.wc = *reinterpret_cast<const uint4*>(rec);
  R.lc = *(reinterpret_cast<const uint4*>(rec + 4) + lane);
  R.e = *(reinterpret_cast<const uint4*>(rec + 4 + 128) + lane);
#pragma unroll
  for (int g = 0; g < 4; g++) R.e2[g] = *(reinterpret_cast<const uint4*>(rec + 4 + 256 + 128 * g) + lane);
}

template <int V>
__global__ void __launch_bounds__(256, 1) lk(unsigned long long* out, int iters) {
  extern __shared__ __align__(16) uint32_t sm[];
  uint32_t* S = sm;                       // 2048-word state
  uint32_t* area = sm + 2048;             // NLAY layer records
  uint32_t* topb = area + NLAY * (16 + 8 * REC_WORDS);
  uint64_t* mb = reinterpret_cast<uint64_t*>(topb + 16);
  const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (uint32_t i = tid; i < 2048; i += 256) S[i] = i * 2654435761u;
  for (uint32_t i = tid; i < NLAY * (16 + 8 * REC_WORDS); i += 256) {
    uint32_t h = i * 2246822519u;
    // leaf entries: word < 2048 byte offsets (<<5) | rot
    area[i] = ((h >> 7) & 0x1FFCu) << 3 | (h & 31u);
  }
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"((uint32_t)__cvta_generic_to_shared(mb)));
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"((uint32_t)__cvta_generic_to_shared(mb)));
  }
  __syncthreads();
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(S);
  Regs R, R2;
  load_rec(area, 0, R);
  load_rec(area, 1, R2);
  uint32_t acc = 0;
  unsigned long long t0 = 0;
  for (int it = 0; it < iters; it++) {
    if (it == 16) t0 = clock64();
    // ---- exec: sparse gather of 4 leaves
    uint32_t v = 0;
    const uint32_t q[4] = {R.e.x, R.e.y, R.e.z, R.e.w};
#pragma unroll
    for (int k = 0; k < 4; k++) {
      uint32_t s;
      asm volatile("ld.shared.u32 %0, [%1];" : "=r"(s) : "r"(sb + ((q[k] >> 5) & 0x1FFCu)));
      v |= __funnelshift_l(s, s, q[k]) & (1u << (k * 7));
    }
    if (V == 5) {   // 16 more sparse leaves (SPARSE entry format: addr e >> 16, rot e, pos e >> 8)
      uint32_t w0 = 0, w1 = 0, w2 = 0, w3 = 0;
#pragma unroll
      for (int g = 0; g < 4; g++) {
        const uint32_t qq[4] = {R.e2[g].x, R.e2[g].y, R.e2[g].z, R.e2[g].w};
        uint32_t s4[4];
#pragma unroll
        for (int k = 0; k < 4; k++)
          asm volatile("ld.shared.u32 %0, [%1];" : "=r"(s4[k]) : "r"(sb + ((qq[k] >> 16) & 0x1FFCu)));
        w0 |= __funnelshift_l(s4[0], s4[0], qq[0]) & __funnelshift_l(1u, 1u, qq[0] >> 8);
        w1 |= __funnelshift_l(s4[1], s4[1], qq[1]) & __funnelshift_l(1u, 1u, qq[1] >> 8);
        w2 |= __funnelshift_l(s4[2], s4[2], qq[2]) & __funnelshift_l(1u, 1u, qq[2] >> 8);
        w3 |= __funnelshift_l(s4[3], s4[3], qq[3]) & __funnelshift_l(1u, 1u, qq[3] >> 8);
      }
      v |= (w0 | w1) | (w2 | w3);
    }
    const uint32_t P = fold5(v, R.lc.x, R.lc.y, R.lc.z);
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(sb + 4 * (1024 + tid)), "r"(P) : "memory");
    const uint32_t u = __ballot_sync(0xFFFFFFFFu, (P >> 30) & 1u);
    const uint32_t Pw = fold5(u, R.wc.x, R.wc.y, R.wc.z);
    if (lane == 0) {
      asm volatile("st.shared.u32 [%0], %1;" ::"r"(sb + 4 * (1536 + warp)), "r"(Pw) : "memory");
      if (V >= 2) topb[warp] = (Pw >> 30) & 1u;
    }
    if (V >= 2 && warp != 0) asm volatile("bar.arrive 1, 256;" ::: "memory");
    acc += P;

    // ---- next records
    if (V == 3) {
      uint32_t done = 0;
      while (!done)
        asm volatile("{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
                     : "=r"(done) : "r"((uint32_t)__cvta_generic_to_shared(mb)), "r"(0u) : "memory");
    }
    if (V >= 1 && V != 4) load_rec(area, (it + 1) % NLAY, R);
    if (V == 4) { R = R2; load_rec(area, (it + 2) % NLAY, R2); }
    if (V >= 2 && warp == 0) {
      asm volatile("bar.sync 1, 256;" ::: "memory");
      if (lane == 0) {
        uint32_t t8 = 0;
#pragma unroll
        for (int w = 0; w < 8; w++) t8 |= topb[w] << w;
        asm volatile("st.shared.u32 [%0], %1;" ::"r"(sb + 4 * 1600), "r"((t8 ^ R.hd.z) & (t8 >> 4)) : "memory");
      }
    }
    __syncthreads();
  }
  unsigned long long t1 = clock64();
  if (tid == 0 && blockIdx.x == 0) out[0] = (t1 - t0) / (iters - 16);
  if (acc == 0x12345u) out[1] = acc;
}

template <int V>
void run(const char* name, unsigned long long* d, int sms) {
  const int smem = (2048 + NLAY * (16 + 8 * REC_WORDS) + 16) * 4 + 16;
  cudaFuncSetAttribute(lk<V>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  lk<V><<<sms, 256, smem>>>(d, 100);
  lk<V><<<sms, 256, smem>>>(d, 2016);
  cudaDeviceSynchronize();
  unsigned long long h = 0;
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("V%d %-60s %6llu clk/layer (%s)\n", V, name, h, cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  unsigned long long* d;
  cudaMalloc(&d, 16);
  run<0>("gather4 + fold5 + ballot + fold5 + wo + syncthreads", d, sms);
  run<1>("+ next records from smem (4 x LDS.128)", d, sms);
  run<2>("+ levels 11-13 hand-off", d, sms);
  run<3>("+ mbarrier try_wait per layer", d, sms);
  run<4>("V2 with records two layers ahead", d, sms);
  run<5>("V2 + 16 more sparse leaves per thread (20 total)", d, sms);
  return 0;
}
