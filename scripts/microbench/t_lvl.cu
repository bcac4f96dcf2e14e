// t_lvl microbenchmarks: the per-level synchronisation
// latency that bounds dependency-bound triangles, measured on the box.
//   1. intra-CTA bar.sync loop (NC threads)
//   2. bar.sync + a shared-memory x chain (ld.shared -> DFMA -> st.shared), as
//      one level of the chain kernel does
//   3. (2) + one global store per row (the chain kernel's xs write)
//   4. cross-SM flag ping-pong through L2 (strong relaxed loads/stores):
//      the dependency latency the sync-free kernel pays per level
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o t_lvl t_lvl.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_bar(int iters, long long* out) {
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) asm volatile("bar.sync 1, %0;" ::"r"(blockDim.x) : "memory");
  if (threadIdx.x == 0) out[0] = clock64() - t0;
}

template <bool STG>
__global__ void k_chain(int iters, long long* out, double* g) {
  __shared__ double xw[4096];
  const int tid = threadIdx.x, n = blockDim.x;
  for (int i = tid; i < 4096; i += n) xw[i] = 1.0 + i * 1e-9;
  __syncthreads();
  const int a0 = (tid * 7 + 3) & 4095, a1 = (tid * 13 + 5) & 4095;
  double v0 = 0.25, v1 = 0.125;
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    double acc = 0.5 - v0 * xw[(a0 + i) & 4095] - v1 * xw[(a1 + i) & 4095];
    const int w = (tid + 2048 + i) & 4095;
    xw[w] = acc;
    if (STG) g[(size_t)i * n + tid] = acc;
    asm volatile("bar.sync 1, %0;" ::"r"(n) : "memory");
  }
  if (tid == 0) out[0] = clock64() - t0;
}

__device__ __forceinline__ int ld_relaxed(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(int* p, int v) {
  asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// two CTAs (different SMs): CTA 0 writes i+1 when it sees i on flag B, CTA 1
// answers on flag A -- one hop = one dependent level of a sync-free solve
__global__ void k_pingpong(int iters, int* fa, int* fb, long long* out) {
  if (threadIdx.x != 0) return;
  long long t0 = clock64();
  if (blockIdx.x == 0) {
    for (int i = 0; i < iters; ++i) {
      st_relaxed(fa, 2 * i + 1);
      while (ld_relaxed(fb) != 2 * i + 1) {
      }
    }
    out[0] = clock64() - t0;
  } else {
    for (int i = 0; i < iters; ++i) {
      while (ld_relaxed(fa) != 2 * i + 1) {
      }
      st_relaxed(fb, 2 * i + 1);
    }
  }
}

int main2();
int main() {
  long long* d_out;
  double* g;
  int *fa, *fb;
  cudaMalloc(&d_out, 64);
  cudaMalloc(&g, 64ull << 20);
  cudaMalloc(&fa, 256);
  cudaMalloc(&fb, 256);
  long long h;
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int iters = 20000;
  for (int nt : {64, 128, 256, 512, 1024}) {
    k_bar<<<1, nt>>>(iters, d_out);
    cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
    double bar = (double)h / iters;
    k_chain<false><<<1, nt>>>(iters, d_out, g);
    cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
    double ch = (double)h / iters;
    k_chain<true><<<1, nt>>>(1000, d_out, g);
    cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
    double chg = (double)h / 1000;
    printf("threads %4d: bar.sync %6.1f cyc | smem chain+bar %6.1f cyc | +STG %6.1f cyc\n", nt, bar, ch, chg);
  }
  cudaMemset(fa, 0, 256);
  cudaMemset(fb, 0, 256);
  k_pingpong<<<2, 32>>>(10000, fa, fb, d_out);
  cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
  printf("cross-SM ping-pong: %.1f cycles per hop (%.3f us at %d MHz nominal)\n", (double)h / 20000,
         (double)h / 20000 / (clk / 1000.0), clk / 1000);
  cudaError_t e = cudaDeviceSynchronize();
  printf("status %s\n", cudaGetErrorString(e));
  return main2();
}

// ---- steps toward the ELL chain kernel, to attribute its per-level cost ----
// B: per-level bounds read from smem + per-row operand prefetch from smem
//    (slot, value x2, b) before the barrier, then LDS x -> 2 DFMA -> STS/STG
// C: B + a producer warp that keeps streaming 64 KB bulk copies into a separate
//    smem buffer (TMA writes competing for the shared-memory port)
__device__ __forceinline__ uint32_t saddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <bool TMA>
__global__ void k_ellish(int iters, long long* out, double* g, const char* src) {
  extern __shared__ __align__(128) unsigned char sm[];
  double* xw = (double*)sm;                 // 4096 + 2
  int* lp = (int*)(sm + 4098 * 8);          // 1024
  int* idx = lp + 1024;                     // 2 x 2048
  double* val = (double*)(idx + 4096);      // 2 x 2048
  double* bb = val + 4096;                  // 2048
  unsigned char* tbuf = (unsigned char*)(bb + 2048);  // 65536 bytes TMA target
  uint64_t* bar = (uint64_t*)(tbuf + 65536);
  const int tid = threadIdx.x;
  const int NC = TMA ? blockDim.x - 32 : blockDim.x;
  for (int i = tid; i < 4098; i += blockDim.x) xw[i] = 1.0 + i * 1e-9;
  for (int i = tid; i < 1024; i += blockDim.x) lp[i] = (i * 700) % 2048;
  for (int i = tid; i < 4096; i += blockDim.x) {
    idx[i] = (i * 7 + 1) & 4095;
    val[i] = 0.25;
  }
  for (int i = tid; i < 2048; i += blockDim.x) bb[i] = 0.5;
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(saddr(bar)) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (TMA && tid >= NC) {
    if (tid == NC) {
      uint32_t ph = 0;
      for (int i = 0; i < iters / 4; ++i) {  // ~64 KB per 4 levels
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(saddr(bar)), "r"(65536)
                     : "memory");
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                saddr(tbuf)),
            "l"(src + (size_t)(i % 64) * 65536), "r"(65536), "r"(saddr(bar))
            : "memory");
        uint32_t done = 0;
        while (!done)
          asm volatile(
              "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0,1,0,p;\n}\n"
              : "=r"(done)
              : "r"(saddr(bar)), "r"(ph)
              : "memory");
        ph ^= 1u;
      }
    }
    return;
  }
  long long t0 = clock64();
  int la = 0, lb = 700;
  for (int it = 0; it < iters; ++it) {
    const int i = la + tid, ok = i < lb, ic = ok ? i & 2047 : 0;
    const int s0 = ok ? idx[ic] : 4096, s1 = ok ? idx[2048 + ic] : 4096;
    const double v0 = ok ? val[ic] : 0.0, v1 = ok ? val[2048 + ic] : 0.0, b = ok ? bb[ic] : 0.0;
    la = lp[it & 1023];
    lb = la + 700;
    asm volatile("bar.sync 1, %0;" ::"r"(NC) : "memory");
    double acc = b - v0 * xw[s0] - v1 * xw[s1];
    if (ok) {
      xw[(i + it) & 4095] = acc;
      g[(size_t)(it & 255) * 1024 + tid] = acc;
    }
  }
  if (tid == 0) out[0] = clock64() - t0;
}

int main2() {
  long long* d_out;
  double* g;
  char* src;
  cudaMalloc(&d_out, 64);
  cudaMalloc(&g, 64ull << 20);
  cudaMalloc(&src, 64ull << 20);
  long long h;
  const int smem = 4098 * 8 + 1024 * 4 + 4096 * 4 + 4096 * 8 + 2048 * 8 + 65536 + 64;
  cudaFuncSetAttribute(k_ellish<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k_ellish<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 20000;
  for (int warps : {8, 12, 16, 24}) {
    k_ellish<false><<<1, 32 * warps, smem>>>(iters, d_out, g, src);
    cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
    double b = (double)h / iters;
    k_ellish<true><<<1, 32 * (warps + 1), smem>>>(iters, d_out, g, src);
    cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
    printf("ELL-like level, %2d warps x 1 row: %6.1f cyc | + concurrent TMA 64KB/4 levels: %6.1f cyc\n", warps, b,
           (double)h / iters);
  }
  printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
