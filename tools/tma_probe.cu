// Probe of TMA box layouts the fused group kernel relies on (tools only; informs group.cpp):
// (1) a tensor map whose dims 1.. are PERMUTED (non-monotonic strides) lands the box densely in
// the map's dim order; (2) a box whose dim 0 runs past the tensor's extent is zero-filled there.
// Element i of the 24^4 source tensor holds i; each smem slot is checked against the model.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <vector>

__global__ void k(const __grid_constant__ CUtensorMap map, double *out, int nbytes, int c0, int c1, int c2, int c3) {
  extern __shared__ __align__(1024) unsigned char sm[];
  unsigned char *s = sm + ((1024 - ((unsigned)__cvta_generic_to_shared(sm) & 1023)) & 1023);
  __shared__ unsigned long long bar;
  unsigned b = (unsigned)__cvta_generic_to_shared(&bar);
  unsigned d = (unsigned)__cvta_generic_to_shared(s);
  for (int i = threadIdx.x; i < nbytes / 8; i += blockDim.x) reinterpret_cast<double *>(s)[i] = -1.0;
  asm volatile("fence.proxy.async.shared::cta;\n" ::: "memory");
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(b));
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(b), "r"(nbytes) : "memory");
    asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];\n"
                 ::"r"(d), "l"(&map), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(b) : "memory");
    asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(b) : "memory");
  }
  __syncthreads();
  for (int i = threadIdx.x; i < nbytes / 8; i += blockDim.x) out[i] = reinterpret_cast<double *>(s)[i];
}

int main() {
  void *p = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  auto enc = (PFN_cuTensorMapEncodeTiled_v12000)p;
  const long N = 24;   // source tensor (x0, x1, x2, x3), x0 fastest, value = linear index
  std::vector<double> h(N * N * N * N);
  for (size_t i = 0; i < h.size(); i++) h[i] = (double)i;
  double *dt, *dout;
  cudaMalloc(&dt, h.size() * 8);
  cudaMemcpy(dt, h.data(), h.size() * 8, cudaMemcpyHostToDevice);
  cudaMalloc(&dout, 1 << 20);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  // map dim j -> source dim perm[j]; box per map dim; coordinates per map dim
  struct Cfg { int perm[4]; unsigned box[4]; int crd[4]; const char *name; } cfgs[] = {
      {{0, 2, 1, 3}, {4, 24, 4, 4}, {4, 0, 8, 12}, "dims (x0,x2,x1,x3) box (4,24,4,4) permuted strides"},
      {{0, 2, 1, 3}, {28, 4, 4, 4}, {0, 4, 8, 4}, "dims (x0,x2,x1,x3) box (28,4,4,4): x0 runs past 24 (OOB)"},
  };
  for (auto &c : cfgs) {
    CUtensorMap map;
    cuuint64_t dims[4], strides[3];
    const long sstr[4] = {1, N, N * N, N * N * N};
    for (int j = 0; j < 4; j++) dims[j] = N;
    for (int j = 1; j < 4; j++) strides[j - 1] = 8 * sstr[c.perm[j]];
    cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = enc(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, dt + 0, dims, strides, c.box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    const int nel = c.box[0] * c.box[1] * c.box[2] * c.box[3];
    k<<<1, 128, 32 * 1024>>>(map, dout, nel * 8, c.crd[0], c.crd[1], c.crd[2], c.crd[3]);
    cudaError_t le = cudaGetLastError();
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<double> o(nel);
    cudaMemcpy(o.data(), dout, nel * 8, cudaMemcpyDeviceToHost);
    int bad = 0, oob = 0;
    for (int s = 0; s < nel; s++) {
      int b[4], rr = s;
      for (int j = 0; j < 4; j++) { b[j] = rr % c.box[j]; rr /= c.box[j]; }
      long src[4] = {0, 0, 0, 0};
      bool in = true;
      for (int j = 0; j < 4; j++) {
        const long x = c.crd[j] + b[j];
        in &= x < N;
        src[c.perm[j]] = x;
      }
      const double want = in ? (double)(src[0] + N * (src[1] + N * (src[2] + N * src[3]))) : 0.0;
      if (!in) oob++;
      if (o[s] != want) { if (bad < 5) printf("  slot %d got %g want %g\n", s, o[s], want); bad++; }
    }
    printf("%s: encode %d launch %s run %s: %d mismatches of %d (%d OOB slots)\n", c.name, (int)r,
           cudaGetErrorString(le), cudaGetErrorString(e), bad, nel, oob);
  }
  return 0;
}
