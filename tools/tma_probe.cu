// Minimal TMA probe: encode a 4D map and load one box; prints the result.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "../paper_conf_sc_valero_laravgr23_b200/csrc/mrlbm_kernels.cuh"
using namespace mr;
__global__ void probe(const __grid_constant__ CUtensorMap tmap, double* out, int c0, int c1, int c3) {
  extern __shared__ __align__(128) unsigned char sm[];
  double* st = (double*)sm;
  uint64_t* bar = (uint64_t*)(sm + 32768);
  if (threadIdx.x == 0) { mbar_init(bar, 1); fence_barrier_init(); }
  __syncthreads();
  if (threadIdx.x == 0) { mbar_expect_tx(bar, 128*1*6*8); tma_load_4d(st, &tmap, bar, c0, c1, 0, c3); }
  mbar_wait(bar, 0);
  for (int i = threadIdx.x; i < 128*6; i += blockDim.x) out[i] = st[i];
}
typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main() {
  int nA = 131, nB = 1, M = 6, P = 5, pitch = 144;
  size_t n = (size_t)P*M*nB*pitch;
  double* buf; cudaMalloc(&buf, n*8);
  double* h = (double*)malloc(n*8); for (size_t i=0;i<n;i++) h[i]=i; cudaMemcpy(buf,h,n*8,cudaMemcpyHostToDevice);
  double* out; cudaMalloc(&out, 128*6*8);
  void* p=nullptr; cudaDriverEntryPointQueryResult q;
  cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  printf("entry %d q %d p %p\n", (int)e, (int)q, p);
  alignas(64) CUtensorMap map;
  cuuint64_t dims[4] = {(cuuint64_t)nA, (cuuint64_t)nB, (cuuint64_t)M, (cuuint64_t)P};
  cuuint64_t str[3] = {(cuuint64_t)pitch*8, (cuuint64_t)nB*pitch*8, (cuuint64_t)M*nB*pitch*8};
  cuuint32_t box[4] = {128, 1, 6, 1}, es[4] = {1,1,1,1};
  CUresult r = ((Enc)p)(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, buf, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode %d\n", (int)r);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 40000);
  int cs[4][2] = {{0,0},{100,0},{0,1},{-1,0}};
  for (auto& cc : cs) { int c0 = cc[0];
    probe<<<1,128,40000>>>(map, out, c0, cc[1], 1);
    e = cudaDeviceSynchronize();
    printf("c0=%d c1=%d launch: %s\n", c0, cc[1], cudaGetErrorString(e));
    if (e) return 1;
    double o[768]; cudaMemcpy(o, out, sizeof(o), cudaMemcpyDeviceToHost);
    printf("  out[0..3] %g %g %g %g  out[30] %g out[31] %g out[40] %g out[128] %g\n", o[0], o[1], o[2], o[3], o[30], o[31], o[40], o[128]);
  }
  return 0;
}
