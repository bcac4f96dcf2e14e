// Single-warp level-step microbenchmark for the strand wavefront kernel
// (tri_wave): cycles per group as features are added to the loop body.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o wave_loop wave_loop.cu
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__device__ __forceinline__ double lds_v(uint32_t a) {
  double v;
  asm volatile("ld.volatile.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ double lds_p(uint32_t a) {
  double v;
  asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts_v(uint32_t a, double v) { asm volatile("st.volatile.shared.f64 [%0], %1;" ::"r"(a), "d"(v)); }
__device__ __forceinline__ void stg_r(double* p, double v) { asm volatile("st.relaxed.gpu.global.f64 [%0], %1;" ::"l"(p), "d"(v)); }
__device__ __forceinline__ void stg_w(double* p, double v) { asm volatile("st.global.f64 [%0], %1;" ::"l"(p), "d"(v)); }
__device__ __forceinline__ bool is_sent(double v) { return __double_as_longlong(v) == (long long)0x7FF4000000000BADull; }

// F bits: 1 operand loads from smem (words/vals/b), 2 sentinel vote, 4 STG relaxed, 8 STG weak,
// 16 push (mapa + st.shared::cluster to own CTA), 32 volatile x loads (else plain), 64 syncwarp
template <int F>
__global__ void k_loop(int iters, long long* out, double* g) {
  __shared__ double xw[1024];
  __shared__ uint32_t wd[2][1024];
  __shared__ double vv[2][1024];
  __shared__ double bb[1024];
  const int lane = threadIdx.x;
  for (int i = lane; i < 1024; i += 32) {
    xw[i] = 1.0 + i * 1e-9;
    wd[0][i] = (i + 1024 - 32) & 1023;
    wd[1][i] = (i + 1024 - 31) & 1023;
    vv[0][i] = 0.25;
    vv[1][i] = 0.125;
    bb[i] = 0.5;
  }
  __syncwarp();
  const uint32_t xs = (uint32_t)__cvta_generic_to_shared(xw);
  long long t0 = clock64();
  uint32_t w0 = lane, w1 = lane + 1;
  double v0 = 0.25, v1 = 0.125, b = 0.5;
  for (int i = 0; i < iters; ++i) {
    const int r = (i * 32 + lane) & 1023;
    double x0, x1;
    if (F & 32) {
      x0 = lds_v(xs + (w0 << 3));
      x1 = lds_v(xs + (w1 << 3));
    } else {
      x0 = lds_p(xs + (w0 << 3));
      x1 = lds_p(xs + (w1 << 3));
    }
    uint32_t nw0 = w0, nw1 = w1;
    double nv0 = v0, nv1 = v1, nb = b;
    if (F & 1) {
      const int rn = ((i + 1) * 32 + lane) & 1023;
      nw0 = wd[0][rn];
      nw1 = wd[1][rn];
      nv0 = vv[0][rn];
      nv1 = vv[1][rn];
      nb = bb[rn];
    } else {
      nw0 = (r + 1024 - 32 + 32) & 1023;
      nw1 = (r + 1024 - 31 + 32) & 1023;
    }
    if (F & 2) {
      bool pend = is_sent(x0) | is_sent(x1);
      while (__any_sync(0xffffffffu, pend)) {
        x0 = lds_v(xs + (w0 << 3));
        pend = is_sent(x0);
      }
    }
    double acc = fma(-v0, x0, b);
    acc = fma(-v1, x1, acc);
    sts_v(xs + (r << 3), acc);
    if (F & 128) {  // speculative: a sentinel operand makes acc a NaN
      if (acc != acc) {
        do {
          x0 = lds_v(xs + (w0 << 3));
          x1 = lds_v(xs + (w1 << 3));
        } while (is_sent(x0) | is_sent(x1));
        acc = fma(-v1, x1, fma(-v0, x0, b));
        sts_v(xs + (r << 3), acc);
      }
    }
    if (F & 256) {
      if (is_sent(x0) | is_sent(x1)) {
        do {
          x0 = lds_v(xs + (w0 << 3));
          x1 = lds_v(xs + (w1 << 3));
        } while (is_sent(x0) | is_sent(x1));
        acc = fma(-v1, x1, fma(-v0, x0, b));
        sts_v(xs + (r << 3), acc);
      }
    }
    if (F & 4) stg_r(g + ((i * 32 + lane) & ((1 << 20) - 1)), acc);
    if (F & 8) stg_w(g + ((i * 32 + lane) & ((1 << 20) - 1)), acc);
    if (F & 16) {
      if (lane == 0) {
        uint32_t ra;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(xs + 8u * 1023), "r"(0));
        asm volatile("st.relaxed.cluster.shared::cluster.f64 [%0], %1;" ::"r"(ra), "d"(acc) : "memory");
      }
    }
    if (F & 64) __syncwarp();
    w0 = nw0; w1 = nw1; v0 = nv0; v1 = nv1; b = nb;
  }
  if (lane == 0) out[F & 127] = clock64() - t0 + (F > 127 ? 0 : 0);
}

template <int F>
void run(int iters, long long* d, double* g, const char* name) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(1);
  cfg.blockDim = dim3(32);
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 1;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, k_loop<F>, iters, d, g);
  long long h[128];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  printf("%-48s F=%3d: %7.1f cycles/group\n", name, F, (double)h[F & 127] / iters);
}

int main_hop();
int main() {
  main_hop();
  long long* d;
  double* g;
  cudaMalloc(&d, 128 * 8);
  cudaMalloc(&g, 8 << 20);
  const int it = 100000;
  run<64>(it, d, g, "chain (plain LDS) + syncwarp");
  run<96>(it, d, g, "chain (volatile LDS) + syncwarp");
  run<97>(it, d, g, "+ operand loads");
  run<99>(it, d, g, "+ operand loads + vote");
  run<103>(it, d, g, "+ operand loads + vote + STG relaxed");
  run<107>(it, d, g, "+ operand loads + vote + STG weak");
  run<115>(it, d, g, "+ ... + push (DSMEM, no STG)");
  run<119>(it, d, g, "+ ... + push + STG relaxed");
  run<32>(it, d, g, "chain (volatile) no syncwarp");
  run<97 + 128>(it, d, g, "+ operand loads + NaN check");
  run<97 + 128 + 4 + 16>(it, d, g, "+ operand loads + NaN check + STG + push");
  run<97 + 256>(it, d, g, "+ operand loads + per-lane sentinel branch");
  run<97 + 256 + 4 + 16>(it, d, g, "+ operand loads + sentinel branch + STG + push");
  printf("status %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}

// ---- hop latency: ping-pong of a value between two warps that poll their
// own shared memory; the partner writes it there (same CTA: st.shared;
// other CTA of the cluster: mapa + st.shared::cluster, weak or relaxed.cluster)
template <int MODE>  // 0 same CTA STS, 1 DSMEM relaxed.cluster, 2 DSMEM weak, 3 DSMEM volatile
__global__ void k_hop(int iters, long long* out) {
  __shared__ double box[2];
  uint32_t rank;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
  const int w = MODE == 0 ? threadIdx.x / 32 : (int)rank;  // player id
  const int lane = threadIdx.x & 31;
  if (threadIdx.x < 2) box[threadIdx.x] = -1.0;
  __syncthreads();
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (MODE != 0 && threadIdx.x >= 32) return;
  const uint32_t mybox = (uint32_t)__cvta_generic_to_shared(&box[w]);
  const uint32_t other = (uint32_t)__cvta_generic_to_shared(&box[1 - w]);
  uint32_t remote;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(other), "r"(1 - rank));
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    if (w == 1 || i > 0) {  // wait for value i
      double v;
      do {
        asm volatile("ld.volatile.shared.f64 %0, [%1];" : "=d"(v) : "r"(mybox));
      } while (v != (double)(2 * i + (w == 1 ? 0 : -1)) && !(w == 0 && v == (double)(2 * i - 1)));
    }
    const double nv = (double)(2 * i + w);
    if (lane == 0) {
      if (MODE == 0) asm volatile("st.volatile.shared.f64 [%0], %1;" ::"r"(other), "d"(nv));
      if (MODE == 1) asm volatile("st.relaxed.cluster.shared::cluster.f64 [%0], %1;" ::"r"(remote), "d"(nv) : "memory");
      if (MODE == 2) asm volatile("st.shared::cluster.f64 [%0], %1;" ::"r"(remote), "d"(nv) : "memory");
      if (MODE == 3) asm volatile("st.volatile.shared::cluster.f64 [%0], %1;" ::"r"(remote), "d"(nv) : "memory");
    }
    __syncwarp();
  }
  if (w == 0 && lane == 0) out[100 + MODE] = clock64() - t0;
}

template <int MODE>
void run_hop(int iters, long long* d, const char* name) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(MODE == 0 ? 1 : 2);
  cfg.blockDim = dim3(MODE == 0 ? 64 : 32);
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = MODE == 0 ? 1 : 2;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, k_hop<MODE>, iters, d);
  cudaError_t e2 = cudaDeviceSynchronize();
  long long h[128];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  printf("hop %-40s: %7.1f cycles per one-way hop (%s/%s)\n", name, (double)h[100 + MODE] / iters / 2,
         cudaGetErrorString(e), cudaGetErrorString(e2));
}

int main_hop() {
  long long* d;
  cudaMalloc(&d, 128 * 8);
  run_hop<0>(20000, d, "same CTA, st.volatile.shared");
  run_hop<1>(20000, d, "DSMEM st.relaxed.cluster");
  run_hop<2>(20000, d, "DSMEM st weak");
  run_hop<3>(20000, d, "DSMEM st.volatile");
  return 0;
}
