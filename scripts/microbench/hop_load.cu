// Cross-SM flag hop latency (st.relaxed.gpu -> ld.relaxed.gpu through L2)
// while other warps poll memory the way sync-free triangles do (debug
// microbenchmark for DESIGN.md sec. 5.3).
//   block 0 and block 1 (different SMs) ping-pong a flag 20000 times;
//   blocks 2.. run `lw` polling warps each: strong loads of random words of a
//   16 MB array (or one hot word), optionally __nanosleep between polls,
//   until the ping-pong ends.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 hop_load.cu -o hop_load
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>

__device__ __forceinline__ int ld_relaxed(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_relaxed(int* p, int v) {
  asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__global__ void k(int iters, int* fa, int* fb, volatile int* stop, const int* arr, int mask, int hot, int sleep_ns,
                  long long* out, unsigned long long* polls) {
  if (blockIdx.x < 2) {
    if (threadIdx.x != 0) return;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      if (blockIdx.x == 0) {
        st_relaxed(fa, 2 * i + 1);
        while (ld_relaxed(fb) != 2 * i + 1) {
        }
      } else {
        while (ld_relaxed(fa) != 2 * i + 1) {
        }
        st_relaxed(fb, 2 * i + 1);
      }
    }
    if (blockIdx.x == 0) {
      out[0] = clock64() - t0;
      *stop = 1;
    }
    return;
  }
  unsigned h = (blockIdx.x * blockDim.x + threadIdx.x) * 2654435761u;
  unsigned long long n = 0;
  int acc = 0;
  while (!*stop) {
    h = h * 1664525u + 1013904223u;
    acc += ld_relaxed(arr + (hot ? 0 : (h & mask)));
    if (sleep_ns) __nanosleep(sleep_ns);
    ++n;
  }
  if (acc == 12345) polls[1] = 1;
  atomicAdd(polls, n);
}

int main(int argc, char** argv) {
  int* f;
  cudaMalloc(&f, 1024);
  int* arr;
  const int N = 1 << 22;
  cudaMalloc(&arr, N * 4);
  cudaMemset(arr, 0, N * 4);
  int* stop;
  cudaMalloc(&stop, 4);
  long long* out;
  cudaMalloc(&out, 8);
  unsigned long long* polls;
  cudaMalloc(&polls, 16);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  const int iters = 20000;
  int loads[] = {0, 512, 2048, 4096, 8192};
  for (int hot = 0; hot < 2; ++hot)
    for (int sl : {0, 100, 400})
      for (int lw : loads) {
        if (hot && sl) continue;
        cudaMemset(f, 0, 1024);
        cudaMemset(stop, 0, 4);
        cudaMemset(polls, 0, 16);
        const int blocks = 2 + (lw + 7) / 8;
        k<<<blocks, 256>>>(iters, f, f + 64, stop, arr, N - 1, hot, sl, out, polls);
        cudaError_t e = cudaDeviceSynchronize();
        long long h = 0;
        unsigned long long np = 0;
        cudaMemcpy(&h, out, 8, cudaMemcpyDeviceToHost);
        cudaMemcpy(&np, polls, 8, cudaMemcpyDeviceToHost);
        const double ns = (double)h / (2.0 * iters) / (clk / 1e6);
        const double secs = (double)h / (clk * 1e3);
        std::printf("%s load_warps=%5d sleep=%3d ns: hop %.0f cycles = %.0f ns; loads %.1f G/s %s\n",
                    hot ? "HOT " : "rand", lw ? ((lw + 7) / 8) * 8 : 0, sl, (double)h / (2.0 * iters), ns,
                    np / secs / 1e9, e == cudaSuccess ? "" : cudaGetErrorString(e));
      }
  return 0;
}
