// Micro-benchmark: one layer's leaf gather (dense16 instruction mix: u16
// entries rot | word<<5, rotl + mask-or per leaf) for 8192 leaves spread over
// NT threads (LPT leaves each), then a 1-STS write-out and a block barrier.
// Answers: is the gather issue-, LDS- or latency-bound, and does spreading it
// over more warps help?  1 CTA per SM, grid = #SMs, clocks per layer on CTA 0.
// Build/run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ug scripts/ubench_gather.cu && /tmp/ug
#include <cstdio>
#include <cstdint>
#include <vector>

template <int NT, int LPT, bool kConflictFree>
__global__ void __launch_bounds__(NT, 1) gk(const uint32_t* __restrict__ ent, unsigned long long* out, int iters) {
  __shared__ __align__(16) uint32_t S[2048];
  const uint32_t tid = threadIdx.x;
  for (uint32_t i = tid; i < 2048; i += NT) S[i] = i * 2654435761u;
  uint32_t q[LPT / 2];
#pragma unroll
  for (int j = 0; j < LPT / 2; j++) {
    uint32_t e = ent[(blockIdx.x * NT + tid) * (LPT / 2) + j];
    if (kConflictFree) e = (e & 0xFFE0FFE0u & ~0xFF80FF80u) | (((tid & 31) << 5) | ((tid & 31) << 21)) | (e & 0x001F001Fu);
    q[j] = e;
  }
  __syncthreads();
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(S);
  unsigned long long t0 = 0;
  uint32_t acc = 0;
  for (int it = 0; it < iters; it++) {
    if (it == 8) t0 = clock64();
    uint32_t a[4] = {0u, 0u, 0u, 0u};
#pragma unroll
    for (int j = 0; j < LPT / 2; j++) {
      uint32_t lo, hi;
      asm volatile("ld.shared.u32 %0, [%1];" : "=r"(lo) : "r"(base + ((q[j] >> 3) & 0x1FFCu)));
      asm volatile("ld.shared.u32 %0, [%1];" : "=r"(hi) : "r"(base + ((q[j] >> 19) & 0x1FFCu)));
      a[j & 3] |= (__funnelshift_l(lo, lo, q[j]) & (1u << (2 * j))) |
                  (__funnelshift_l(hi, hi, q[j] >> 16) & (1u << (2 * j + 1)));
    }
    const uint32_t v = (a[0] | a[1]) | (a[2] | a[3]);
    acc += v;
    // write-out into the state the next layer reads
    asm volatile("st.shared.u32 [%0], %1;" ::"r"(base + 4 * ((tid * 8 + it) & 2047)), "r"(v) : "memory");
    __syncthreads();
  }
  unsigned long long t1 = clock64();
  if (tid == 0 && blockIdx.x == 0) out[0] = (t1 - t0) / (iters - 8);
  if (acc == 0x12345u) out[1] = acc;
}

template <int NT, int LPT, bool CF>
void run(const char* name, const uint32_t* d_ent, unsigned long long* d, int sms) {
  unsigned long long h = 0;
  gk<NT, LPT, CF><<<sms, NT>>>(d_ent, d, 40);
  gk<NT, LPT, CF><<<sms, NT>>>(d_ent, d, 1008);
  cudaDeviceSynchronize();
  cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
  printf("%-40s %6llu clk/layer  (%s)\n", name, h, cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  std::vector<uint32_t> h(sms * 1024 * 16);
  uint64_t x = 88172645463325252ull;
  for (auto& v : h) {
    x ^= x << 13; x ^= x >> 7; x ^= x << 17;
    const uint32_t w0 = (x >> 3) & 2047, r0 = x & 31, w1 = (x >> 20) & 2047, r1 = (x >> 40) & 31;
    v = (r0 | w0 << 5) | ((r1 | w1 << 5) << 16);
  }
  uint32_t* d_ent;
  unsigned long long* d;
  cudaMalloc(&d_ent, h.size() * 4);
  cudaMalloc(&d, 16);
  cudaMemcpy(d_ent, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  run<256, 32, false>("256 thr x 32 leaves, random words", d_ent, d, sms);
  run<256, 32, true>("256 thr x 32 leaves, conflict-free", d_ent, d, sms);
  run<512, 16, false>("512 thr x 16 leaves, random words", d_ent, d, sms);
  run<512, 16, true>("512 thr x 16 leaves, conflict-free", d_ent, d, sms);
  run<1024, 8, false>("1024 thr x 8 leaves, random words", d_ent, d, sms);
  run<1024, 8, true>("1024 thr x 8 leaves, conflict-free", d_ent, d, sms);
  run<256, 8, false>("256 thr x 8 leaves (light layer)", d_ent, d, sms);
  run<256, 2, false>("256 thr x 2 leaves (lightest)", d_ent, d, sms);
  return 0;
}
