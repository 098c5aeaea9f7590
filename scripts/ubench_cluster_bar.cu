// Micro-benchmark: grid barrier round trip among G co-resident CTAs (1 per
// SM, 256 threads), flat flags (gem_runtime.cu grid_sync) vs a two-level
// barrier on thread-block clusters: hardware cluster barrier, then the
// cluster leaders exchange flags (one per cluster), then the cluster barrier
// again.  Also reports how many clusters of each size can be co-resident.
// Build/run: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ucb scripts/ubench_cluster_bar.cu && /tmp/ucb
#include <cooperative_groups.h>
#include <cstdint>
#include <cstdio>
#include <vector>

#define NT 256
#define STRIDE 16

__device__ __forceinline__ unsigned long long ld_acq(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_rel(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t cluster_id_x() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t nclusters_x() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(r));
  return r;
}

// MODE 0: flat flags; 1: cluster barrier + leader flags + cluster barrier
template <int MODE>
__global__ void __launch_bounds__(NT, 1) k(unsigned long long* bar, unsigned long long* out, int iters) {
  const uint32_t tid = threadIdx.x;
  unsigned long long ep = 0;
  unsigned long long t0 = 0;
  for (int it = 0; it < iters; it++) {
    if (it == 8) t0 = clock64();
    ep++;
    if (MODE == 0) {
      __syncthreads();
      if (tid == 0) st_rel(bar + (size_t)blockIdx.x * STRIDE, ep);
      for (uint32_t f = tid; f < gridDim.x; f += NT)
        while (ld_acq(bar + (size_t)f * STRIDE) < ep) {}
      __syncthreads();
    } else {
      asm volatile("barrier.cluster.arrive.release.aligned;\n" ::: "memory");
      asm volatile("barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
      const uint32_t nc = nclusters_x(), cid = cluster_id_x();
      if (cluster_rank() == 0) {
        if (tid == 0) st_rel(bar + (size_t)cid * STRIDE, ep);
        for (uint32_t f = tid; f < nc; f += NT)
          while (ld_acq(bar + (size_t)f * STRIDE) < ep) {}
        __syncthreads();
      }
      asm volatile("barrier.cluster.arrive.release.aligned;\n" ::: "memory");
      asm volatile("barrier.cluster.wait.acquire.aligned;\n" ::: "memory");
    }
  }
  unsigned long long t1 = clock64();
  if (tid == 0 && blockIdx.x == 0) out[0] = (t1 - t0) / (iters - 8);
}

template <int MODE>
void run(int G, int cs, unsigned long long* d_bar, unsigned long long* d_out) {
  cudaMemset(d_bar, 0, 4096 * STRIDE * 8);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(G);
  cfg.blockDim = dim3(NT);
  cfg.dynamicSmemBytes = 180 * 1024;   // one CTA per SM, like the word kernel
  cudaFuncSetAttribute(k<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, 180 * 1024);
  if (cs > 8) cudaFuncSetAttribute(k<MODE>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  cudaLaunchAttribute at[2];
  int na = 0;
  at[na].id = cudaLaunchAttributeCooperative;
  at[na].val.cooperative = 1;
  na++;
  if (cs > 1) {
    at[na].id = cudaLaunchAttributeClusterDimension;
    at[na].val.clusterDim.x = cs;
    at[na].val.clusterDim.y = 1;
    at[na].val.clusterDim.z = 1;
    na++;
  }
  cfg.attrs = at;
  cfg.numAttrs = na;
  int ncl = -1;
  if (cs > 1) cudaOccupancyMaxActiveClusters(&ncl, k<MODE>, &cfg);
  cudaError_t e = cudaLaunchKernelEx(&cfg, k<MODE>, d_bar, d_out, 2008);
  cudaError_t e2 = cudaDeviceSynchronize();
  unsigned long long h = 0;
  cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
  printf("mode %d grid %4d cluster %2d (max active clusters %3d): %6llu clk/barrier  (%s / %s)\n", MODE, G, cs, ncl, h,
         cudaGetErrorString(e), cudaGetErrorString(e2));
}

int main() {
  unsigned long long *d_bar, *d_out;
  cudaMalloc(&d_bar, 4096 * STRIDE * 8);
  cudaMalloc(&d_out, 64);
  for (int G : {128, 136, 144}) run<0>(G, 1, d_bar, d_out);
  for (int cs : {2, 4, 8})
    for (int G : {128, 136, 144}) {
      if (G % cs) continue;
      run<1>(G, cs, d_bar, d_out);
    }
  run<1>(128, 16, d_bar, d_out);
  return 0;
}
