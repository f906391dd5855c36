#include <cstdio>
#include "/root/repo/paper_conf_sc_valero_laravgr23_b200/csrc/mrlbm_kernels.cuh"
using namespace mr;
__global__ void k(double* out) {
  double m[6] = {0.01, 0.03, -0.02, 0.001, 0.0005, -0.0003};
  double A[9]; double f[9];
  collide_coeffs<0, true, double>(m, 0.3, A);
  reconstruct<0, true, double>(A, f);
  for (int i=0;i<9;i++) out[i]=A[i];
  for (int i=0;i<9;i++) out[9+i]=f[i];
}
int main(){ double* d; cudaMalloc(&d, 18*8); k<<<1,1>>>(d); double h[18]; cudaMemcpy(h,d,sizeof(h),cudaMemcpyDeviceToHost); for(int i=0;i<18;i++) printf("%g ", h[i]); printf("\n"); }
