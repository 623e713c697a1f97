// tools/peaks.cu — B200 microbenchmarks that set the FP64 roofline denominators
// (SURVEY §7 step 4): DFMA vs DMMA (mma.sync f64 shapes) throughput, HBM
// read / write / copy bandwidth, and the SM clock seen under FP64 load.
// Also checks the DMMA fragment layouts the libtc kernels rely on.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o peaks tools/peaks.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>
#include <vector>
#include <cmath>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

__device__ unsigned long long g_clk[2];

// ---- DFMA: 16 independent chains per thread --------------------------------
template <int CH>
__global__ void k_dfma(double* out, int iters, double s) {
  double a[CH];
#pragma unroll
  for (int i = 0; i < CH; i++) a[i] = threadIdx.x * 1e-3 + i;
  long long t0 = clock64();
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int i = 0; i < CH; i++) a[i] = fma(a[i], s, 1e-7);
  }
  long long t1 = clock64();
  double r = 0;
#pragma unroll
  for (int i = 0; i < CH; i++) r += a[i];
  if (r == 1234.5) out[0] = r;
  if (blockIdx.x == 0 && threadIdx.x == 0) { g_clk[0] = t1 - t0; }
}

// ---- DMMA m8n8k4: ACC independent accumulators per warp ---------------------
template <int ACC>
__global__ void k_dmma884(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 - threadIdx.x * 1e-4;
  double c[ACC][2];
#pragma unroll
  for (int i = 0; i < ACC; i++) { c[i][0] = i; c[i][1] = -i; }
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int i = 0; i < ACC; i++)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                   : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
  }
  double r = 0;
#pragma unroll
  for (int i = 0; i < ACC; i++) r += c[i][0] + c[i][1];
  if (r == 1234.5) out[0] = r;
}

template <int ACC>
__global__ void k_dmma1688(double* out, int iters) {
  double a0 = threadIdx.x * 1e-3, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3;
  double b0 = 1.0 - threadIdx.x * 1e-4, b1 = b0 + 0.5;
  double c[ACC][4];
#pragma unroll
  for (int i = 0; i < ACC; i++) { c[i][0] = i; c[i][1] = -i; c[i][2] = 1; c[i][3] = 2; }
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int i = 0; i < ACC; i++)
      asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
                   : "+d"(c[i][0]), "+d"(c[i][1]), "+d"(c[i][2]), "+d"(c[i][3])
                   : "d"(a0), "d"(a1), "d"(a2), "d"(a3), "d"(b0), "d"(b1));
  }
  double r = 0;
#pragma unroll
  for (int i = 0; i < ACC; i++) r += c[i][0] + c[i][1] + c[i][2] + c[i][3];
  if (r == 1234.5) out[0] = r;
}

template <int ACC>
__global__ void k_dmma16816(double* out, int iters) {
  double a[8], b[4];
#pragma unroll
  for (int i = 0; i < 8; i++) a[i] = threadIdx.x * 1e-3 + i;
#pragma unroll
  for (int i = 0; i < 4; i++) b[i] = 1.0 - threadIdx.x * 1e-4 + i;
  double c[ACC][4];
#pragma unroll
  for (int i = 0; i < ACC; i++) { c[i][0] = i; c[i][1] = -i; c[i][2] = 1; c[i][3] = 2; }
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int i = 0; i < ACC; i++)
      asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};\n"
                   : "+d"(c[i][0]), "+d"(c[i][1]), "+d"(c[i][2]), "+d"(c[i][3])
                   : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                     "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]));
  }
  double r = 0;
#pragma unroll
  for (int i = 0; i < ACC; i++) r += c[i][0] + c[i][1] + c[i][2] + c[i][3];
  if (r == 1234.5) out[0] = r;
}

// ---- fragment layout probe: one warp, m16n8k8 with A[m][k] = m*100+k, B[k][n] = (k==n0?)...
// Writes what each lane holds after D = A*B with A = identity-ish probes, so the host can
// check the documented layout: A a0:(g,t) a1:(g+8,t) a2:(g,t+4) a3:(g+8,t+4); B b0:(t,g) b1:(t+4,g);
// C c0:(g,2t) c1:(g,2t+1) c2:(g+8,2t) c3:(g+8,2t+1).
__global__ void k_layout1688(const double* A /*16x8 row-major*/, const double* B /*8x8 k-major rows*/,
                             double* D /*16x8*/) {
  int lane = threadIdx.x, g = lane >> 2, t = lane & 3;
  double a0 = A[g * 8 + t], a1 = A[(g + 8) * 8 + t], a2 = A[g * 8 + t + 4], a3 = A[(g + 8) * 8 + t + 4];
  double b0 = B[t * 8 + g], b1 = B[(t + 4) * 8 + g];
  double c0 = 0, c1 = 0, c2 = 0, c3 = 0;
  asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};\n"
               : "+d"(c0), "+d"(c1), "+d"(c2), "+d"(c3)
               : "d"(a0), "d"(a1), "d"(a2), "d"(a3), "d"(b0), "d"(b1));
  D[g * 8 + 2 * t] = c0; D[g * 8 + 2 * t + 1] = c1;
  D[(g + 8) * 8 + 2 * t] = c2; D[(g + 8) * 8 + 2 * t + 1] = c3;
}
__global__ void k_layout884(const double* A /*8x4*/, const double* B /*4x8*/, double* D /*8x8*/) {
  int lane = threadIdx.x, g = lane >> 2, t = lane & 3;
  double a0 = A[g * 4 + t], b0 = B[t * 8 + g], c0 = 0, c1 = 0;
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(c0), "+d"(c1) : "d"(a0), "d"(b0));
  D[g * 8 + 2 * t] = c0; D[g * 8 + 2 * t + 1] = c1;
}

// ---- HBM ----------------------------------------------------------------------
__global__ void k_copy(const double4* __restrict__ a, double4* __restrict__ b, size_t n) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x, st = (size_t)gridDim.x * blockDim.x;
  for (; i < n; i += st) b[i] = a[i];
}
__global__ void k_read(const double4* __restrict__ a, double* out, size_t n) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x, st = (size_t)gridDim.x * blockDim.x;
  double s = 0;
  for (; i < n; i += st) { double4 v = a[i]; s += v.x + v.y + v.z + v.w; }
  if (s == 1234.5) out[0] = s;
}
__global__ void k_write(double4* __restrict__ b, size_t n) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x, st = (size_t)gridDim.x * blockDim.x;
  for (; i < n; i += st) b[i] = make_double4(1, 2, 3, 4);
}
__global__ void k_write_f64(double* __restrict__ b, size_t n) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x, st = (size_t)gridDim.x * blockDim.x;
  for (; i < n; i += st) b[i] = 1.0;
}

template <typename F>
static float time_ms(F f, int reps) {
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  f(); CK(cudaDeviceSynchronize());
  CK(cudaEventRecord(a));
  for (int i = 0; i < reps; i++) f();
  CK(cudaEventRecord(b)); CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return ms / reps;
}

int main() {
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  int sms = p.multiProcessorCount;
  int clk_khz = 0; cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
  double* out; CK(cudaMalloc(&out, 64));
  printf("{\"gpu\": \"%s\", \"sms\": %d, \"l2_bytes\": %d, \"smem_optin\": %zu, \"clock_khz_attr\": %d",
         p.name, sms, p.l2CacheSize, p.sharedMemPerBlockOptin, clk_khz);

  // DFMA
  {
    const int iters = 20000, thr = 256, blocks = sms * 8;
    float ms = time_ms([&] { k_dfma<16><<<blocks, thr>>>(out, iters, 0.999999); }, 5);
    double fl = 2.0 * 16 * iters * (double)thr * blocks;
    unsigned long long clk; CK(cudaMemcpyFromSymbol(&clk, g_clk, 8));
    printf(", \"dfma_tflops\": %.3f, \"dfma_ms\": %.3f, \"dfma_sm_mhz_est\": %.0f", fl / ms / 1e9, ms,
           clk / (ms * 1e3));
  }
  // DMMA shapes
  {
    const int iters = 4000, thr = 256;
    for (int occ : {4, 8}) {
      int blocks = sms * occ;
      float ms = time_ms([&] { k_dmma884<8><<<blocks, thr>>>(out, iters); }, 5);
      double fl = 2.0 * 8 * 8 * 4 * 8 * iters * (double)(thr / 32) * blocks;
      printf(", \"dmma884_occ%d_tflops\": %.3f", occ, fl / ms / 1e9);
      ms = time_ms([&] { k_dmma1688<8><<<blocks, thr>>>(out, iters); }, 5);
      fl = 2.0 * 16 * 8 * 8 * 8 * iters * (double)(thr / 32) * blocks;
      printf(", \"dmma1688_occ%d_tflops\": %.3f", occ, fl / ms / 1e9);
      ms = time_ms([&] { k_dmma16816<4><<<blocks, thr>>>(out, iters); }, 5);
      fl = 2.0 * 16 * 8 * 16 * 4 * iters * (double)(thr / 32) * blocks;
      printf(", \"dmma16816_occ%d_tflops\": %.3f", occ, fl / ms / 1e9);
    }
    // latency-ish: one warp per SM with 1 and 4 accumulators
    float ms1 = time_ms([&] { k_dmma884<1><<<sms, 32>>>(out, iters); }, 3);
    printf(", \"dmma884_1acc_1warp_ns_per_mma\": %.2f", ms1 * 1e6 / iters);
    float ms4 = time_ms([&] { k_dmma884<4><<<sms, 32>>>(out, iters); }, 3);
    printf(", \"dmma884_4acc_1warp_ns_per_mma\": %.2f", ms4 * 1e6 / (4.0 * iters));
    float ms8 = time_ms([&] { k_dmma1688<1><<<sms, 32>>>(out, iters); }, 3);
    printf(", \"dmma1688_1acc_1warp_ns_per_mma\": %.2f", ms8 * 1e6 / iters);
  }
  // layout probes
  {
    std::vector<double> hA(16 * 8), hB(8 * 8), hD(16 * 8);
    for (int i = 0; i < 16 * 8; i++) hA[i] = (i * 7) % 13 - 6;
    for (int i = 0; i < 64; i++) hB[i] = (i * 5) % 11 - 5;
    double *dA, *dB, *dD; CK(cudaMalloc(&dA, 1024)); CK(cudaMalloc(&dB, 1024)); CK(cudaMalloc(&dD, 1024));
    CK(cudaMemcpy(dA, hA.data(), 16 * 8 * 8, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dB, hB.data(), 64 * 8, cudaMemcpyHostToDevice));
    k_layout1688<<<1, 32>>>(dA, dB, dD); CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(hD.data(), dD, 16 * 8 * 8, cudaMemcpyDeviceToHost));
    int bad = 0;
    for (int m = 0; m < 16; m++) for (int n = 0; n < 8; n++) {
      double s = 0; for (int k = 0; k < 8; k++) s += hA[m * 8 + k] * hB[k * 8 + n];
      if (s != hD[m * 8 + n]) bad++;
    }
    printf(", \"layout1688_bad\": %d", bad);
    // 884: A 8x4 row-major, B 4x8
    for (int i = 0; i < 32; i++) hA[i] = (i * 7) % 13 - 6;
    CK(cudaMemcpy(dA, hA.data(), 32 * 8, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dB, hB.data(), 32 * 8, cudaMemcpyHostToDevice));
    k_layout884<<<1, 32>>>(dA, dB, dD); CK(cudaDeviceSynchronize());
    CK(cudaMemcpy(hD.data(), dD, 64 * 8, cudaMemcpyDeviceToHost));
    bad = 0;
    for (int m = 0; m < 8; m++) for (int n = 0; n < 8; n++) {
      double s = 0; for (int k = 0; k < 4; k++) s += hA[m * 4 + k] * hB[k * 8 + n];
      if (s != hD[m * 8 + n]) bad++;
    }
    printf(", \"layout884_bad\": %d", bad);
  }
  // HBM
  {
    size_t bytes = (size_t)4 << 30, n4 = bytes / 32;
    double4 *a, *b; CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes));
    CK(cudaMemset(a, 0, bytes));
    int blocks = sms * 8, thr = 512;
    float ms = time_ms([&] { k_copy<<<blocks, thr>>>(a, b, n4); }, 10);
    printf(", \"hbm_copy_gbs\": %.1f", 2.0 * bytes / ms / 1e6);
    ms = time_ms([&] { k_read<<<blocks, thr>>>(a, out, n4); }, 10);
    printf(", \"hbm_read_gbs\": %.1f", 1.0 * bytes / ms / 1e6);
    ms = time_ms([&] { k_write<<<blocks, thr>>>(b, n4); }, 10);
    printf(", \"hbm_write_gbs\": %.1f", 1.0 * bytes / ms / 1e6);
    ms = time_ms([&] { k_write_f64<<<blocks, thr>>>((double*)b, bytes / 8); }, 10);
    printf(", \"hbm_write_f64_gbs\": %.1f", 1.0 * bytes / ms / 1e6);
    ms = time_ms([&] { CK(cudaMemsetAsync(b, 0, bytes)); }, 10);
    printf(", \"memset_gbs\": %.1f", 1.0 * bytes / ms / 1e6);
    CK(cudaFree(a)); CK(cudaFree(b));
  }
  printf("}\n");
  return 0;
}
