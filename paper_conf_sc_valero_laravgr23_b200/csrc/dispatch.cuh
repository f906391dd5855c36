// dispatch.cuh -- template instances of the kernels behind a plain function
// table (Variant / StVariant), so that each lattice compiles in its own
// translation unit (var_d2q9.cu, var_d3q19.cu, var_d3q27.cu, var_st.cu) and the
// host code (mrlbm.cu) selects one at mrlbm_create.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>

#include "../../include/mrlbm.h"
#include "mrlbm_kernels.cuh"
#include "st_kernels.cuh"
#include "step3d.cuh"

namespace mrd {

using mr::StepArgs;

struct Variant {
    int TA, TB, S, BW;
    int CL;            // CTAs per cluster along B (3D; 1 = no clusters)
    size_t smem;
    void (*step)(const CUtensorMap &, const StepArgs &, dim3, cudaStream_t);
    void (*step_push)(const CUtensorMap &, const StepArgs &, dim3, cudaStream_t); // P2P boundary layers (or null)
    const void *kernel_fn_push;
    void (*set)(const double *, void *, mr::GridArgs, cudaStream_t);
    void (*get)(const void *, double *, mr::GridArgs, cudaStream_t);
    void (*pops)(const void *, double *, mr::GridArgs, double, cudaStream_t);
    void (*finite)(const void *, mr::GridArgs, int *, cudaStream_t);
    void (*fd)(const mr::FdArgs &, long long, cudaStream_t);
    const void *kernel_fn;
};

inline int grid_for(long long n) { return (int)std::min<long long>((n + 255) / 256, 148LL * 16); }

// one launch of a step-kernel instance: grid (tiles A, tiles B, segments);
// CL > 1 launches clusters of CL CTAs along grid.y (cudaLaunchKernelEx)
template <class KF> inline void launch_step(KF kernel, int CL, int threads, size_t smem, const CUtensorMap &map,
                                            const StepArgs &a, dim3 grid, cudaStream_t st)
{
    if (CL <= 1) {
        kernel<<<grid, threads, smem, st>>>(map, a);
        return;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = dim3(threads, 1, 1);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 1;
    attr[0].val.clusterDim.y = CL;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, kernel, map, a);
}

template <int LAT, bool REC, typename Real, int TA, int TB, int S, int MINB, bool WITH_PUSH = false, int CL = 1>
Variant make_variant()
{
    using L = mr::Lattice<LAT>;
    using SM = mr::StepSmem<LAT, Real, TA, TB, S, CL>;
    Variant v;
    v.TA = TA;
    v.TB = TB;
    v.S = S;
    v.BW = SM::BW;
    v.CL = CL;
    v.smem = SM::bytes;
    v.kernel_fn = (const void *)mr::mrlbm_step_kernel<LAT, REC, Real, TA, TB, S, MINB, false, CL>;
    v.step = [](const CUtensorMap &map, const StepArgs &a, dim3 grid, cudaStream_t st) {
        launch_step(mr::mrlbm_step_kernel<LAT, REC, Real, TA, TB, S, MINB, false, CL>, CL, TA * TB, SM::bytes, map, a,
                    grid, st);
    };
    v.step_push = nullptr;
    v.kernel_fn_push = nullptr;
    if constexpr (WITH_PUSH) {
        v.kernel_fn_push = (const void *)mr::mrlbm_step_kernel<LAT, REC, Real, TA, TB, S, MINB, true, CL>;
        v.step_push = [](const CUtensorMap &map, const StepArgs &a, dim3 grid, cudaStream_t st) {
            launch_step(mr::mrlbm_step_kernel<LAT, REC, Real, TA, TB, S, MINB, true, CL>, CL, TA * TB, SM::bytes, map,
                        a, grid, st);
        };
    }
    v.set = [](const double *in, void *buf, mr::GridArgs g, cudaStream_t st) {
        mr::set_moments_kernel<L::M, Real><<<grid_for((long long)g.nA * g.nB * g.nC), 256, 0, st>>>(
            in, (Real *)buf, g);
    };
    v.get = [](const void *buf, double *out, mr::GridArgs g, cudaStream_t st) {
        mr::get_moments_kernel<L::M, Real><<<grid_for((long long)g.nA * g.nB * g.nC), 256, 0, st>>>(
            (const Real *)buf, out, g);
    };
    v.pops = [](const void *buf, double *out, mr::GridArgs g, double omega, cudaStream_t st) {
        mr::populations_kernel<LAT, REC, Real><<<grid_for((long long)g.nA * g.nB * g.nC), 256, 0, st>>>(
            (const Real *)buf, out, g, omega);
    };
    v.finite = [](const void *buf, mr::GridArgs g, int *flag, cudaStream_t st) {
        mr::finite_kernel<L::M, Real><<<grid_for((long long)g.nA * g.nB * g.nC), 256, 0, st>>>(
            (const Real *)buf, g, flag);
    };
    v.fd = [](const mr::FdArgs &a, long long nodes, cudaStream_t st) {
        mr::fd_face_kernel<LAT, Real><<<grid_for(nodes), 256, 0, st>>>(a);
    };
    return v;
}

// the paired 3D kernel (step3d.cuh): same Variant table, TA = 32, no clusters
template <int LAT, bool REC, typename Real, int TB, int S, int MINB, bool WITH_PUSH = false, bool SPLIT = false,
          bool ONEBODY = false>
Variant make_variant3()
{
    using SM = mr::Step3Smem<LAT, Real, TB, S>;
    Variant v = make_variant<LAT, REC, Real, 32, TB, S, MINB, false, 1>(); // side kernels
    v.BW = SM::BW;
    v.smem = SM::bytes;
    v.kernel_fn = (const void *)mr::mrlbm_step3_kernel<LAT, REC, Real, TB, S, MINB, false, SPLIT, ONEBODY>;
    v.step = [](const CUtensorMap &map, const StepArgs &a, dim3 grid, cudaStream_t st) {
        mr::mrlbm_step3_kernel<LAT, REC, Real, TB, S, MINB, false, SPLIT, ONEBODY><<<grid, 32 * TB, SM::bytes, st>>>(map, a);
    };
    v.step_push = nullptr;
    v.kernel_fn_push = nullptr;
    if constexpr (WITH_PUSH) {
        v.kernel_fn_push = (const void *)mr::mrlbm_step3_kernel<LAT, REC, Real, TB, S, MINB, true, SPLIT, ONEBODY>;
        v.step_push = [](const CUtensorMap &map, const StepArgs &a, dim3 grid, cudaStream_t st) {
            mr::mrlbm_step3_kernel<LAT, REC, Real, TB, S, MINB, true, SPLIT, ONEBODY><<<grid, 32 * TB, SM::bytes, st>>>(map, a);
        };
    }
    return v;
}

// ---- distribution representation (ST)
struct StVariant {
    int BX;
    void (*step)(const mr::StArgs &, dim3, cudaStream_t);
    void (*set)(const double *, void *, mr::StGrid, cudaStream_t);
    void (*set_pops)(const double *, void *, mr::StGrid, cudaStream_t);
    void (*get)(const void *, double *, mr::StGrid, cudaStream_t);
    void (*pops)(const void *, double *, mr::StGrid, double, double, cudaStream_t);
    void (*finite)(const void *, mr::StGrid, int *, cudaStream_t);
    const void *kernel_fn;
};

template <int LAT, int COLL, typename Real> StVariant make_st()
{
    constexpr int BX = 128;
    StVariant v;
    v.BX = BX;
    v.kernel_fn = (const void *)mr::st_step_kernel<LAT, COLL, Real, BX>;
    v.step = [](const mr::StArgs &a, dim3 grid, cudaStream_t st) {
        mr::st_step_kernel<LAT, COLL, Real, BX><<<grid, BX, 0, st>>>(a);
    };
    v.set = [](const double *in, void *buf, mr::StGrid g, cudaStream_t st) {
        mr::st_set_moments_kernel<LAT, Real><<<grid_for((long long)g.nx * g.ny * g.nz), 256, 0, st>>>(in, (Real *)buf, g);
    };
    v.set_pops = [](const double *in, void *buf, mr::StGrid g, cudaStream_t st) {
        mr::st_set_populations_kernel<LAT, Real><<<grid_for((long long)g.nx * g.ny * g.nz), 256, 0, st>>>(in, (Real *)buf, g);
    };
    v.get = [](const void *buf, double *out, mr::StGrid g, cudaStream_t st) {
        mr::st_get_moments_kernel<LAT, Real><<<grid_for((long long)g.nx * g.ny * g.nz), 256, 0, st>>>((const Real *)buf, out, g);
    };
    v.pops = [](const void *buf, double *out, mr::StGrid g, double omega, double inv_tau, cudaStream_t st) {
        mr::st_populations_kernel<LAT, COLL, Real><<<grid_for((long long)g.nx * g.ny * g.nz), 256, 0, st>>>(
            (const Real *)buf, out, g, omega, inv_tau);
    };
    v.finite = [](const void *buf, mr::StGrid g, int *flag, cudaStream_t st) {
        mr::st_finite_kernel<LAT, Real><<<grid_for((long long)g.nx * g.ny * g.nz), 256, 0, st>>>((const Real *)buf, g, flag);
    };
    return v;
}


// per-lattice tables (one translation unit each)
Variant pick_d2q9(bool rec, bool f32, int tile, int cluster);
Variant pick_d3q19(bool rec, bool f32, int tile, int cluster);
Variant pick_d3q27(bool rec, bool f32, int tile, int cluster);
StVariant select_st(int lat, int coll, int prec);
// moments (eqs 1-3) of dense fp64 populations [Q][N] -> dense fp64 [M][N] (set_populations)
void moments_of_populations(int lat, double *pops, double *mom, int nx, int rows, cudaStream_t st);

} // namespace mrd
