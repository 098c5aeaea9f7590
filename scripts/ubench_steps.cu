// Micro-benchmark: cost of one barrier-separated step of word-level AND ops
// (one signal per 32-bit word, the LAN2 lane-program model) for a SINGLE
// stream, 1 CTA per SM.  Each step: every thread runs M ops
// (two dependent-free LDS, inversions, LOP3, STS), then __syncthreads.
// Answers: clk per step for 256 / 512 / 1024 threads and M = 1 / 2, with op
// words resident in shared memory (SM) or streamed from L2 into registers.
// Build/run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/us scripts/ubench_steps.cu && /tmp/us
#include <cstdint>
#include <cstdio>
#include <vector>
#include <random>

#define NW 8192     // state words
#define NSTEPS 64

// op: x = a_byte | b_byte << 16, y = dst_byte | ia << 30 | ib << 31 (dst 0 = none)
template <int NT, int M, bool OPS_SMEM>
__global__ void __launch_bounds__(NT, 1) k(const uint2* __restrict__ ops, unsigned long long* out, int reps) {
  extern __shared__ __align__(16) uint32_t sm[];
  uint32_t* S = sm;
  uint2* O = reinterpret_cast<uint2*>(sm + NW);
  const uint32_t tid = threadIdx.x;
  for (uint32_t i = tid; i < NW; i += NT) S[i] = i * 2654435761u;
  if (OPS_SMEM)
    for (uint32_t i = tid; i < NSTEPS * M * NT; i += NT) O[i] = ops[blockIdx.x * NSTEPS * M * NT + i];
  __syncthreads();
  const uint32_t sb = (uint32_t)__cvta_generic_to_shared(S);
  const uint32_t ob = (uint32_t)__cvta_generic_to_shared(O);
  unsigned long long t0 = 0;
  for (int r = 0; r < reps; r++) {
    if (r == 2) t0 = clock64();
    const uint2* g = ops + blockIdx.x * NSTEPS * M * NT + tid;
#pragma unroll 4
    for (int s = 0; s < NSTEPS; s++) {
      uint2 o[M];
#pragma unroll
      for (int j = 0; j < M; j++) {
        if (OPS_SMEM) {
          asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(o[j].x), "=r"(o[j].y) : "r"(ob + 8 * ((s * M + j) * NT + tid)));
        } else {
          o[j] = __ldg(g + (s * M + j) * NT);
        }
      }
      uint32_t a[M], b[M];
#pragma unroll
      for (int j = 0; j < M; j++) {
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(a[j]) : "r"(sb + (o[j].x & 0xFFFFu)));
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(b[j]) : "r"(sb + (o[j].x >> 16)));
      }
#pragma unroll
      for (int j = 0; j < M; j++) {
        const uint32_t v = (a[j] ^ (o[j].y >> 30)) & (b[j] ^ (o[j].y >> 31));
        if (o[j].y & 0xFFFFu) asm volatile("st.shared.u32 [%0], %1;" ::"r"(sb + (o[j].y & 0xFFFFu)), "r"(v) : "memory");
      }
      __syncthreads();
    }
  }
  unsigned long long t1 = clock64();
  if (tid == 0) out[blockIdx.x] = (t1 - t0) / ((unsigned long long)(reps - 2) * NSTEPS);
}

template <int NT, int M, bool OS>
void run(const char* name, const uint2* d_ops, unsigned long long* d_out, int G) {
  const size_t smem = NW * 4 + (OS ? (size_t)NSTEPS * M * NT * 8 : 0);
  cudaFuncSetAttribute(k<NT, M, OS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  k<NT, M, OS><<<G, NT, smem>>>(d_ops, d_out, 4);
  k<NT, M, OS><<<G, NT, smem>>>(d_ops, d_out, 40);
  cudaError_t e = cudaDeviceSynchronize();
  std::vector<unsigned long long> h(G);
  cudaMemcpy(h.data(), d_out, G * 8, cudaMemcpyDeviceToHost);
  double m = 0;
  for (auto x : h) m += x;
  printf("%-34s %6.0f clk/step  (%s)\n", name, m / G, cudaGetErrorString(e));
}

int main() {
  const int G = 148;
  const int maxops = NSTEPS * 2 * 1024;
  std::mt19937 rng(3);
  std::vector<uint2> ops((size_t)G * maxops);
  for (auto& o : ops) {
    // word addresses in [1, NW): random (conflicts as they come)
    const uint32_t a = 1 + rng() % (NW - 1), b = 1 + rng() % (NW - 1), d = 1 + rng() % (NW - 1);
    o.x = (a * 4) | ((b * 4) << 16);
    o.y = (d * 4) | ((rng() & 3u) << 30);
  }
  uint2* d_ops;
  unsigned long long* d_out;
  cudaMalloc(&d_ops, ops.size() * 8);
  cudaMemcpy(d_ops, ops.data(), ops.size() * 8, cudaMemcpyHostToDevice);
  cudaMalloc(&d_out, G * 8);
  run<256, 1, false>("256 thr, M=1, ops from L2", d_ops, d_out, G);
  run<256, 1, true>("256 thr, M=1, ops in smem", d_ops, d_out, G);
  run<256, 2, true>("256 thr, M=2, ops in smem", d_ops, d_out, G);
  run<256, 4, true>("256 thr, M=4, ops in smem", d_ops, d_out, G);
  run<512, 1, true>("512 thr, M=1, ops in smem", d_ops, d_out, G);
  run<512, 2, true>("512 thr, M=2, ops in smem", d_ops, d_out, G);
  run<1024, 1, true>("1024 thr, M=1, ops in smem", d_ops, d_out, G);
  run<128, 1, true>("128 thr, M=1, ops in smem", d_ops, d_out, G);
  run<128, 2, true>("128 thr, M=2, ops in smem", d_ops, d_out, G);
  run<64, 1, true>("64 thr, M=1, ops in smem", d_ops, d_out, G);
  run<32, 1, true>("32 thr (1 warp, bar), M=1, smem", d_ops, d_out, G);
  return 0;
}
