// ubench_pipes.cu -- measured issue throughput / latency of the arithmetic the
// 3D step kernels are made of (FFMA vs packed FFMA2, DFMA, DADD) on this B200.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/ubp tools/ubench_pipes.cu
#include <cstdio>
#include <cuda_runtime.h>
#define N_ITER 4096
template <int ILP> __global__ void k_ffma(float *out, float s)
{
    float a[ILP];
    for (int i = 0; i < ILP; i++) a[i] = threadIdx.x + i;
    for (int it = 0; it < N_ITER; it++)
#pragma unroll
        for (int i = 0; i < ILP; i++) a[i] = fmaf(a[i], s, 0.5f);
    float r = 0; for (int i = 0; i < ILP; i++) r += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = r;
}
template <int ILP> __global__ void k_ffma2(float *out, float s)
{
    float2 a[ILP];
    for (int i = 0; i < ILP; i++) a[i] = make_float2(threadIdx.x + i, i);
    const float2 S = make_float2(s, s), H = make_float2(0.5f, 0.5f);
    for (int it = 0; it < N_ITER; it++)
#pragma unroll
        for (int i = 0; i < ILP; i++) a[i] = __ffma2_rn(a[i], S, H);
    float r = 0; for (int i = 0; i < ILP; i++) r += a[i].x + a[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = r;
}
template <int ILP> __global__ void k_dfma(float *out, double s)
{
    double a[ILP];
    for (int i = 0; i < ILP; i++) a[i] = threadIdx.x + i;
    for (int it = 0; it < N_ITER; it++)
#pragma unroll
        for (int i = 0; i < ILP; i++) a[i] = fma(a[i], s, 0.5);
    double r = 0; for (int i = 0; i < ILP; i++) r += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = (float)r;
}
template <int ILP> __global__ void k_dadd(float *out, double s)
{
    double a[ILP];
    for (int i = 0; i < ILP; i++) a[i] = threadIdx.x + i;
    for (int it = 0; it < N_ITER; it++)
#pragma unroll
        for (int i = 0; i < ILP; i++) a[i] = a[i] + s;
    double r = 0; for (int i = 0; i < ILP; i++) r += a[i];
    out[blockIdx.x * blockDim.x + threadIdx.x] = (float)r;
}
template <class K> void run(const char *name, K kern, int ilp, int flops_per_op, int blocks, int threads, float *out)
{
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    kern<<<blocks, threads>>>(out, 1.0000001);
    cudaEventRecord(e0);
    kern<<<blocks, threads>>>(out, 1.0000001);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)blocks * threads * N_ITER * ilp; // thread-level instructions
    int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    double cyc = ms * 1e-3 * clk * 1e3;
    printf("%-8s ILP=%2d blocks=%5d thr=%4d  %.3f ms  warp-inst/clk/SM=%.3f  lanes-op/clk/SM=%.1f  (%.1f Gop/s)\n", name, ilp,
           blocks, threads, ms, ops / 32 / cyc / 148, ops / cyc / 148, ops / ms * 1e-6);
}
int main()
{
    float *out; cudaMalloc(&out, 148 * 64 * 1024 * sizeof(float));
    for (int w : {1, 4, 8, 16}) {
        int blocks = 148, thr = 32 * w;
        run("ffma", k_ffma<1>, 1, 2, blocks, thr, out);
        run("ffma", k_ffma<8>, 8, 2, blocks, thr, out);
        run("ffma2", k_ffma2<1>, 1, 4, blocks, thr, out);
        run("ffma2", k_ffma2<8>, 8, 4, blocks, thr, out);
        run("dfma", k_dfma<1>, 1, 2, blocks, thr, out);
        run("dfma", k_dfma<8>, 8, 2, blocks, thr, out);
        run("dadd", k_dadd<1>, 1, 1, blocks, thr, out);
        run("dadd", k_dadd<8>, 8, 1, blocks, thr, out);
    }
    return 0;
}
