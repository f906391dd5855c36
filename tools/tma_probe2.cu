// TMA probe with arbitrary 4D dims / box / coords (fp64): ./tma_probe2 d0 d1 d2 d3 pitch b0 b1 b2 c0 c1 c3
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include "../paper_conf_sc_valero_laravgr23_b200/csrc/mrlbm_kernels.cuh"
using namespace mr;
__global__ void probe(const __grid_constant__ CUtensorMap tmap, double* out, int c0, int c1, int c3, unsigned bytes) {
  extern __shared__ __align__(128) unsigned char sm[];
  double* st = (double*)sm;
  uint64_t* bar = (uint64_t*)(sm + 65536);
  if (threadIdx.x == 0) { mbar_init(bar, 1); fence_barrier_init(); }
  __syncthreads();
  if (threadIdx.x == 0) { mbar_expect_tx(bar, bytes); tma_load_4d(st, &tmap, bar, c0, c1, 0, c3); }
  mbar_wait(bar, 0);
  if (threadIdx.x == 0) out[0] = st[0];
}
typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main(int argc, char** argv) {
  long d[4]; for (int i=0;i<4;i++) d[i]=atol(argv[1+i]);
  long pitch = atol(argv[5]);
  unsigned bx[3]; for (int i=0;i<3;i++) bx[i]=atoi(argv[6+i]);
  int c0=atoi(argv[9]), c1=atoi(argv[10]), c3=atoi(argv[11]);
  size_t n = (size_t)d[3]*d[2]*d[1]*pitch;
  double* buf; cudaMalloc(&buf, n*8); cudaMemset(buf, 0, n*8);
  double* out; cudaMalloc(&out, 8);
  void* p=nullptr; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  alignas(64) CUtensorMap map;
  cuuint64_t dims[4] = {(cuuint64_t)d[0], (cuuint64_t)d[1], (cuuint64_t)d[2], (cuuint64_t)d[3]};
  cuuint64_t str[3] = {(cuuint64_t)pitch*8, (cuuint64_t)d[1]*pitch*8, (cuuint64_t)d[2]*d[1]*pitch*8};
  cuuint32_t box[4] = {bx[0], bx[1], bx[2], 1}, es[4] = {1,1,1,1};
  CUresult r = ((Enc)p)(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, buf, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 70000);
  probe<<<1,128,70000>>>(map, out, c0, c1, c3, bx[0]*bx[1]*bx[2]*8);
  cudaError_t e = cudaDeviceSynchronize();
  printf("dims %ld %ld %ld %ld pitch %ld box %u %u %u coords %d %d %d: encode %d launch %s\n", d[0],d[1],d[2],d[3],pitch,bx[0],bx[1],bx[2],c0,c1,c3,(int)r,cudaGetErrorString(e));
  return 0;
}
