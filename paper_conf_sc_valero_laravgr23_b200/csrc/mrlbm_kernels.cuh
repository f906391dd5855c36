// mrlbm_kernels.cuh -- the fused sm_100a MR-LBM timestep and its helpers.
//
// One launch = one timestep of the moment representation (Alg. 2,
// P:L185-261): read the moments (rho, u, Pi) of a tile, collide in moment
// space (eq 10; eqs 12-13 for recursive), reconstruct the post-collision
// populations (eq 11 / eq 14), stream them (eq 7) across the CTA through
// shared memory with a one-node halo, apply the boundary
// treatment, recompute the moments of the completed layer (eqs 1-3,
// P:L259) and write them back.  Only moments touch HBM.
//
// B200 design: a CTA owns a (TA-2) x (TB-2) in-plane
// tile (2D: TA-2 x 1) and sweeps a segment of layers along the marching
// axis C.  Per layer a TMA box {TA, TB, M, 1} (tile + halo ring, all M
// moment planes) lands in an S-deep shared-memory ring guarded by mbarriers;
// in-plane moving populations are exchanged through one shared-memory plane;
// populations moving along C never leave the thread: they are accumulated
// into rolling per-layer moment accumulators (layers c-1, c, c+1) held in
// registers, which replaces the paper's (z_t + 2)-layer shared population
// array.  The state is stored shifted (rho - 1, populations f - w_i) for
// precision (R16).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "lattice.cuh"

// rotated 3D sweep in the scalar kernel (see the kernel): default on; measured
// C5 fp64 +9%, C3 fp64 +0.7%; the 2D kernel keeps the plain sweep (C2 -1% / -4.5%
// rotated), profiles/r03/ab10.jsonl
#ifndef MRLBM_ROTATE_SCALAR
#define MRLBM_ROTATE_SCALAR 1
#endif

namespace mr {

enum { BC_PERIODIC = 0, BC_WALL = 1, BC_MOVING = 2, BC_VELOCITY = 3, BC_PRESSURE = 4 };

// Kernel-axis faces: 0 A-, 1 A+, 2 B-, 3 B+, 4 C-, 5 C+.
struct StepArgs {
    const void *src;        // node (0,0) of plane 0 (low ghost plane) of the source buffer
    void *dst;              // same for the destination buffer
    int padA, padB;         // storage pad before node 0 along A / B (TMA box origins must be >= 0)
    int nA, nB, nC;         // local extents (nB = 1 in 2D)
    int pitch;              // elements per A-row
    long long mstride;      // elements between moment planes = nB * pitch
    long long pstride;      // elements between layers         = M * nB * pitch
    int c_begin, c_end;     // owned layers updated by this launch (segments 0 .. nseg1-1 of grid.y)
    int seg_len;            // layers per CTA segment
    int nseg1;              // segments of the first range; grid.y beyond it covers [c2_begin, c2_end)
    int c2_begin, c2_end;   // optional second range (a slab's first and last layer in one launch)
    int tilesA;             // tiles along A
    int tilesB;             // tiles along B (3D)
    int rastG;              // 3D, CL = 1: grid.x = tilesA * tilesB in launch groups of rastG B-tiles (0: grid (A, B))
    int lo_nb, hi_nb;       // 1 if layer -1 / nC exists (periodic wrap or ghost plane)
    int wrapC;              // 1: layer c lives in plane wrap(c)+1 (single-rank periodic C)
    int c_offset;           // global index of local layer 0 (profiles)
    int kind[6];            // face kinds (C faces: WALL/MOVING only at this rank's global ends)
    double uw[6][3];        // wall velocities (physical x, y, z)
    double open_drho[4];    // PRESSURE faces: rho - 1
    double open_u[4][3];    // VELOCITY faces: uniform velocity
    const double *open_prof[4]; // VELOCITY faces: optional [face nodes][D] (global)
    double omega;           // 1 - 1/tau
    // P2P transport (peer memory over NVLink): node (0,0) of the lower / upper
    // neighbour's ghost plane in its copy of this step's destination buffer.
    // Layer 0 / nC-1 of the new state is pushed there as it is finalized, so
    // the halo exchange rides on the stores of the fused step (null: no push)
    void *peer_lo, *peer_hi;
};

// ------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void *p)
{
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_barrier_init()
{
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity)
{
    uint32_t addr = smem_u32(bar);
    asm volatile(
        "{\n"
        ".reg .pred p;\n"
        "WAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
        "@!p bra WAIT_%=;\n"
        "}\n" ::"r"(addr),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_4d(void *dst, const CUtensorMap *map, uint64_t *bar, int c0, int c1,
                                            int c2, int c3)
{
    asm volatile(
        "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], "
        "[%2];" ::"r"(smem_u32(dst)),
        "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
        : "memory");
}
// thread-block clusters (3D kernels with CL > 1): rank in the cluster, the
// cluster-wide barrier (release / acquire: shared-memory stores into a peer
// CTA before the arrive are visible to its threads after the wait), and the
// shared::cluster address of the same smem location in CTA `rank`
__device__ __forceinline__ uint32_t cluster_ctarank()
{
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all()
{
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t mapa_shared(uint32_t addr, uint32_t rank)
{
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
    return r;
}
__device__ __forceinline__ void st_cluster(uint32_t addr, double v)
{
    asm volatile("st.shared::cluster.f64 [%0], %1;" ::"r"(addr), "d"(v) : "memory");
}
__device__ __forceinline__ void st_cluster(uint32_t addr, float v)
{
    asm volatile("st.shared::cluster.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap *map)
{
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

// ------------------------------------------------------------ node algebra
// Collided, scaled Hermite coefficients A'_h of one node (eqs 10, 12, 13 and
// their orders-5/6 extension for D3Q27; recursive a^neq from the pair-sum
// closed form of Malaspinas' recursion, R8):
//   n = 0: rho - 1 (shifted zeroth moment)     n = 1: rho u_a
//   n = 2: omega Pi_ab + (1 - omega) rho u_a u_b           (= Pi*, eq 10)
//   n > 2: rho u^h + omega sum_{pairs p<q} Pneq_{a_p a_q} u^{h - e_{a_p} - e_{a_q}}
// each times hscale(h).  The pair sum is grouped by pair type: (a,a) occurs
// C(h_a, 2) times and (a,b), a < b, h_a h_b times, so every term is one FMA
// against a monomial u^m (m <= (2,2,2)) computed once per node.
// The full tensor bases (D2Q9 / D3Q27 recursive) use the sum-factorised
// reconstruction, which applies the per-axis Hermite scale and the D1Q3
// weights itself; their coefficients carry only tscale(h) = 6^-(#axes with h = 0).
// Reconstruction scheme per variant (and the coefficient scale collide_coeffs
// applies for it):
//   PAIR      D2Q9 projective: even/odd pairing of i and opp(i); coefficients
//             times hscale(h) = prod_a 1/(h_a! c_s^{2 h_a})  (eq 11)
//   TENSOR_W  D2Q9-R, D3Q27-P/R: sum-factorised 1D Hermite synthesis per axis
//             with the D1Q3 weights folded in (their weights are D1Q3
//             products); coefficients times tscale(h) = 6^-(#axes with h = 0)
//   TENSOR_U  D3Q19-P/R: the same synthesis without weights (D3Q19 weights are
//             not products), coefficients times hscale(h) / 36, then
//             f_i = (36 w_i) V(c_i) with 36 w_i in {12, 2, 1}
// Components absent from a basis (projective: n > 2; D3Q19-R: R10) are
// compile-time zeros in the synthesis, and populations a lattice does not
// have are never read, so their arithmetic is removed at compile time.
enum { RECON_PAIR = 0, RECON_TENSOR_W = 1, RECON_TENSOR_U = 2 };
template <int LAT, bool REC> constexpr int recon_kind()
{
    return LAT == LAT_D2Q9 ? (REC ? RECON_TENSOR_W : RECON_PAIR) : (LAT == LAT_D3Q27 ? RECON_TENSOR_W : RECON_TENSOR_U);
}
template <int LAT, bool REC> constexpr bool tensor_recon() { return recon_kind<LAT, REC>() == RECON_TENSOR_W; }
constexpr double tscale(int D, int h0, int h1, int h2)
{
    const int z = (h0 == 0) + (h1 == 0) + (D == 3 && h2 == 0);
    return z == 0 ? 1.0 : (z == 1 ? 1.0 / 6 : (z == 2 ? 1.0 / 36 : 1.0 / 216));
}

template <int LAT, bool REC, typename Real>
__device__ __forceinline__ void collide_coeffs(const Real (&m)[Lattice<LAT>::M], Real omega,
                                               Real (&A)[Basis<LAT, REC>::NH])
{
    using L = Lattice<LAT>;
    using B = Basis<LAT, REC>;
    constexpr int D = L::D;
    const Real drho = m[0];
    const Real rho = Real(1) + drho;
    Real u[3];
    u[0] = m[1];
    u[1] = m[2];
    u[2] = (D == 3) ? m[3] : Real(0);
    const Real omc = Real(1) - omega;
    Real Pn[3][3]; // Pi^neq (eq 8 in moment form: Pi - rho u u)
    Real up[3][3]; // up[a][k] = u_a^k
    if constexpr (REC) {
#pragma unroll
        for (int a = 0; a < D; a++)
#pragma unroll
            for (int b = a; b < D; b++) {
                Pn[a][b] = m[pslot<D>(a, b)] - rho * u[a] * u[b];
                Pn[b][a] = Pn[a][b];
            }
#pragma unroll
        for (int a = 0; a < 3; a++) {
            up[a][0] = Real(1);
            up[a][1] = u[a];
            up[a][2] = u[a] * u[a];
        }
    }
    // u^(m0,m1,m2); factors equal to 1 are dropped at compile time
    auto mono = [&](auto m0c, auto m1c, auto m2c) -> Real {
        constexpr int m0 = decltype(m0c)::value, m1 = decltype(m1c)::value, m2 = decltype(m2c)::value;
        if constexpr (m0 + m1 + m2 == 0) return Real(1);
        else if constexpr (m1 + m2 == 0) return up[0][m0];
        else if constexpr (m0 + m2 == 0) return up[1][m1];
        else if constexpr (m0 + m1 == 0) return up[2][m2];
        else if constexpr (m2 == 0) return up[0][m0] * up[1][m1];
        else if constexpr (m1 == 0) return up[0][m0] * up[2][m2];
        else if constexpr (m0 == 0) return up[1][m1] * up[2][m2];
        else return up[0][m0] * up[1][m1] * up[2][m2];
    };
    using I0 = std::integral_constant<int, 0>;
    constexpr int RK = recon_kind<LAT, REC>();
    const Real omc_rho = omc * rho;
    static_for<0, B::NH>([&](auto hk) {
        constexpr int k = decltype(hk)::value;
        constexpr int h0 = B::h[k][0], h1 = B::h[k][1], h2 = B::h[k][2];
        constexpr int n = h0 + h1 + h2;
        // the coefficient's scale (see recon_kind); it rides on rho, omega and
        // omc * rho, one product per distinct scale shared by every component
        // that has it (omega * sc is loop-invariant)
        constexpr Real sc = Real(RK == RECON_TENSOR_W ? tscale(D, h0, h1, h2)
                                                      : (RK == RECON_TENSOR_U ? hscale(h0, h1, h2) / 36.0
                                                                              : hscale(h0, h1, h2)));
        constexpr int i0 = (h0 > 0) ? 0 : ((h1 > 0) ? 1 : 2);
        Real val;
        if constexpr (n == 0) {
            val = sc == Real(1) ? drho : drho * sc;
        } else if constexpr (n == 1) {
            val = (rho * sc) * u[i0];
        } else if constexpr (n == 2) {
            constexpr int i1 = (h0 == 2) ? 0 : ((h0 == 1) ? ((h1 > 0) ? 1 : 2) : ((h1 == 2) ? 1 : 2));
            val = fma(omega * sc, m[pslot<D>(i0, i1)], (omc_rho * sc) * (u[i0] * u[i1]));
        } else {
            using H0 = std::integral_constant<int, h0>;
            using H1 = std::integral_constant<int, h1>;
            using H2 = std::integral_constant<int, h2>;
            Real aneq = Real(0);
            // (a,a) pairs: C(h_a, 2) = 1 iff h_a == 2
            if constexpr (h0 == 2) aneq = fma(Pn[0][0], mono(I0{}, H1{}, H2{}), aneq);
            if constexpr (h1 == 2) aneq = fma(Pn[1][1], mono(H0{}, I0{}, H2{}), aneq);
            if constexpr (h2 == 2) aneq = fma(Pn[2][2], mono(H0{}, H1{}, I0{}), aneq);
            // (a,b) pairs: h_a h_b of them
            if constexpr (h0 * h1 > 0)
                aneq = fma(Real(h0 * h1) * Pn[0][1],
                           mono(std::integral_constant<int, h0 - 1>{}, std::integral_constant<int, h1 - 1>{}, H2{}), aneq);
            if constexpr (h0 * h2 > 0)
                aneq = fma(Real(h0 * h2) * Pn[0][2],
                           mono(std::integral_constant<int, h0 - 1>{}, H1{}, std::integral_constant<int, h2 - 1>{}), aneq);
            if constexpr (h1 * h2 > 0)
                aneq = fma(Real(h1 * h2) * Pn[1][2],
                           mono(H0{}, std::integral_constant<int, h1 - 1>{}, std::integral_constant<int, h2 - 1>{}), aneq);
            val = fma(omega * sc, aneq, (rho * sc) * mono(H0{}, H1{}, H2{}));
        }
        A[k] = val;
    });
}

// Post-collision coefficients of D3Q19 for the U36 synthesis (synth_p U36, SYN_U36) (eq 10; eqs 12-13 through
// the pair-sum closed form of the recursion, R8), all divided by 36 and with
// no per-component Hermite scale (the synthesis applies it per axis).  With
// r = rho/36, P'_ab = Pi^neq_ab / 36 = Pi_ab/36 - r u_a u_b:
//   order 0: (rho - 1)/36      order 1: r u_a      order 2: Pi*_ab = r u_a u_b + omega P'_ab
//   order 3 (recursive), e.g. (2,1,0): r ux^2 uy + omega (P'xx uy + 2 P'xy ux)
//                                      = uy Pi*_xx + ux R_xy,   R_ab = 2 omega P'_ab
//   order 4, e.g. (2,2,0): r ux^2 uy^2 + omega (P'xx uy^2 + P'yy ux^2 + 4 P'xy ux uy)
//                          = uy a_210 + ux (omega P'yy ux + R_xy uy)
// (the same coefficients collide_coeffs forms term by term, regrouped)
template <bool REC, typename Real>
__device__ __forceinline__ void collide_u36(const Real (&m)[10], Real omega, Real (&A)[Basis<LAT_D3Q19, REC>::NH])
{
    constexpr Real k = Real(1.0 / 36.0);
    const Real drho = m[0];
    const Real r = fma(drho, k, k);
    const Real ux = m[1], uy = m[2], uz = m[3];
    const Real rx = r * ux, ry = r * uy, rz = r * uz;
    const Real rxx = rx * ux, ryy = ry * uy, rzz = rz * uz, rxy = rx * uy, rxz = rx * uz, ryz = ry * uz;
    const Real pxx = fma(m[4], k, -rxx), pyy = fma(m[5], k, -ryy), pzz = fma(m[6], k, -rzz);
    const Real pxy = fma(m[7], k, -rxy), pxz = fma(m[8], k, -rxz), pyz = fma(m[9], k, -ryz);
    A[0] = drho * k;
    A[1] = rx;
    A[2] = ry;
    A[3] = rz;
    if constexpr (REC) {
        const Real oxx = omega * pxx, oyy = omega * pyy, ozz = omega * pzz;
        const Real w2 = omega + omega;
        const Real Rxy = w2 * pxy, Rxz = w2 * pxz, Ryz = w2 * pyz;
        const Real Sxx = rxx + oxx, Syy = ryy + oyy, Szz = rzz + ozz;
        A[4] = Sxx;
        A[5] = Syy;
        A[6] = Szz;
        A[7] = fma(Real(0.5), Rxy, rxy);
        A[8] = fma(Real(0.5), Rxz, rxz);
        A[9] = fma(Real(0.5), Ryz, ryz);
        // basis order (lattice.cuh): 210 201 120 021 102 012 220 202 022
        const Real a210 = fma(uy, Sxx, ux * Rxy), a201 = fma(uz, Sxx, ux * Rxz);
        const Real a120 = fma(ux, Syy, uy * Rxy), a021 = fma(uz, Syy, uy * Ryz);
        const Real a102 = fma(ux, Szz, uz * Rxz), a012 = fma(uy, Szz, uz * Ryz);
        A[10] = a210;
        A[11] = a201;
        A[12] = a120;
        A[13] = a021;
        A[14] = a102;
        A[15] = a012;
        A[16] = fma(ux, fma(oyy, ux, Rxy * uy), uy * a210);
        A[17] = fma(ux, fma(ozz, ux, Rxz * uz), uz * a201);
        A[18] = fma(uy, fma(ozz, uy, Ryz * uz), uz * a021);
    } else {
        A[4] = fma(omega, pxx, rxx);
        A[5] = fma(omega, pyy, ryy);
        A[6] = fma(omega, pzz, rzz);
        A[7] = fma(omega, pxy, rxy);
        A[8] = fma(omega, pxz, rxz);
        A[9] = fma(omega, pyz, ryz);
    }
}

template <int LAT, bool REC> constexpr int hindex(int a, int b, int c)
{
    for (int k = 0; k < Basis<LAT, REC>::NH; k++)
        if (Basis<LAT, REC>::h[k][0] == a && Basis<LAT, REC>::h[k][1] == b && Basis<LAT, REC>::h[k][2] == c) return k;
    return -1;
}

// Weighted 1D Hermite synthesis at c = -1, 0, +1: the per-axis Hermite scale
// hscale(a,b,c) = s(a) s(b) s(c) (s(0) = 1, s(1) = 3, s(2) = 3/2) and the D1Q3
// weight w(0) = 2/3, w(+-1) = 1/6 folded in, for a0 = A0 / 6 (tscale):
//   G(0) = w(0) (A0 - 3/2 A2) = 4 a0 - A2,  G(+-1) = w(1) (A0 + 3 A2 +- 3 A1) = a0 + A2/2 +- A1/2
template <typename Real>
__device__ __forceinline__ void synth3w(Real a0, Real A1, Real A2, Real &gm, Real &g0, Real &gp)
{
    const Real S = fma(Real(0.5), A2, a0);
    g0 = fma(Real(4), a0, -A2);
    gp = fma(Real(0.5), A1, S);
    gm = fma(Real(-0.5), A1, S);
}

// Sum-factorised eq 14 for the full tensor bases {0,1,2}^D (D2Q9 / D3Q27
// recursive): the Hermite-to-population map times w_i is the D-fold tensor
// product of the weighted 1D map above (the weights are D1Q3 products),
// applied axis by axis (z, y, x).  Coefficients arrive scaled by tscale(h).
template <int LAT, typename Real>
__device__ __forceinline__ void reconstruct_tensor(const Real (&A)[Basis<LAT, true>::NH], Real (&f)[Lattice<LAT>::Q])
{
    using L = Lattice<LAT>;
    constexpr int D = L::D;
    Real T[3][3][3]; // [h_x][h_y][c_z + 1]
    static_for<0, 9>([&](auto abk) {
        constexpr int a = decltype(abk)::value / 3, b = decltype(abk)::value % 3;
        constexpr int k0 = hindex<LAT, true>(a, b, 0);
        static_assert(k0 >= 0, "basis component missing");
        if constexpr (D == 3) {
            constexpr int k1 = hindex<LAT, true>(a, b, 1), k2 = hindex<LAT, true>(a, b, 2);
            static_assert(k1 >= 0 && k2 >= 0, "basis component missing");
            synth3w(A[k0], A[k1], A[k2], T[a][b][0], T[a][b][1], T[a][b][2]);
        } else {
            T[a][b][1] = A[k0];
        }
    });
    constexpr int z0 = (D == 3) ? 0 : 1, z1 = (D == 3) ? 3 : 2;
    Real U[3][3][3]; // [h_x][c_y + 1][c_z + 1]
#pragma unroll
    for (int a = 0; a < 3; a++)
#pragma unroll
        for (int zi = z0; zi < z1; zi++) synth3w(T[a][0][zi], T[a][1][zi], T[a][2][zi], U[a][0][zi], U[a][1][zi], U[a][2][zi]);
    Real V[3][3][3]; // [c_x + 1][c_y + 1][c_z + 1]
#pragma unroll
    for (int yi = 0; yi < 3; yi++)
#pragma unroll
        for (int zi = z0; zi < z1; zi++) synth3w(U[0][yi][zi], U[1][yi][zi], U[2][yi][zi], V[0][yi][zi], V[1][yi][zi], V[2][yi][zi]);
    static_for<0, L::Q>([&](auto ik) {
        constexpr int i = decltype(ik)::value;
        constexpr int xi = L::c[i][0] + 1, yi = L::c[i][1] + 1, zi = L::c[i][2] + 1;
        f[i] = V[xi][yi][zi];
    });
}

// ---- 3D sum-factorised synthesis with compile-time absent components.
// One 1D synthesis maps coefficients (x0, x1, x2) of orders 0, 1, 2 along an
// axis to values at c = -1, 0, +1:
//   weighted (TENSOR_W):   g0 = 4 x0 - x2,  g+- = x0 + x2/2 +- x1/2
//   unweighted (TENSOR_U): g0 = x0 - x2,    g+- = x0 + 2 x2 +- x1
// An input that is absent (a compile-time zero) is skipped; an output is
// present if any input it depends on is.
constexpr bool syn_present(int c, bool p0, bool p1, bool p2) { return c == 0 ? (p0 || p2) : (p0 || p1 || p2); }

// U36: unweighted with the per-axis Hermite scale applied here (coefficients
// from collide_u36): g0 = x0 - 3/2 x2, g+- = x0 + 3 x2 +- 3 x1
template <bool W, bool P0, bool P1, bool P2, typename Real, bool U36 = false>
__device__ __forceinline__ void synth_p(Real x0, Real x1, Real x2, Real &gm, Real &g0, Real &gp)
{
    Real S;
    if constexpr (U36 && !W) {
        if constexpr (P0 && P2) { S = fma(Real(3), x2, x0); g0 = fma(Real(-1.5), x2, x0); }
        else if constexpr (P0) { S = x0; g0 = x0; }
        else if constexpr (P2) { S = Real(3) * x2; g0 = Real(-1.5) * x2; }
        if constexpr (P1 && (P0 || P2)) { gp = fma(Real(3), x1, S); gm = fma(Real(-3), x1, S); }
        else if constexpr (P1) { gp = Real(3) * x1; gm = Real(-3) * x1; }
        else if constexpr (P0 || P2) { gp = S; gm = S; }
        else { gp = gm = Real(0); }
        if constexpr (!(P0 || P2)) g0 = Real(0);
    } else if constexpr (W) {
        if constexpr (P0 && P2) { S = fma(Real(0.5), x2, x0); g0 = fma(Real(4), x0, -x2); }
        else if constexpr (P0) { S = x0; g0 = Real(4) * x0; }
        else if constexpr (P2) { S = Real(0.5) * x2; g0 = -x2; }
        if constexpr (P1 && (P0 || P2)) { gp = fma(Real(0.5), x1, S); gm = fma(Real(-0.5), x1, S); }
        else if constexpr (P1) { gp = Real(0.5) * x1; gm = Real(-0.5) * x1; }
        else if constexpr (P0 || P2) { gp = S; gm = S; }
        else { gp = gm = Real(0); } // absent (never read)
        if constexpr (!(P0 || P2)) g0 = Real(0);
    } else {
        if constexpr (P0 && P2) { S = fma(Real(2), x2, x0); g0 = x0 - x2; }
        else if constexpr (P0) { S = x0; g0 = x0; }
        else if constexpr (P2) { S = x2 + x2; g0 = -x2; }
        if constexpr (P1 && (P0 || P2)) { gp = S + x1; gm = S - x1; }
        else if constexpr (P1) { gp = x1; gm = -x1; }
        else if constexpr (P0 || P2) { gp = S; gm = S; }
        else { gp = gm = Real(0); } // absent (never read)
        if constexpr (!(P0 || P2)) g0 = Real(0);
    }
}

// presence of T[a][b][cz] (after the z synthesis) and U[a][cy][cz] (after y)
template <int LAT, bool REC> constexpr bool presT(int a, int b, int cz)
{
    return syn_present(cz, hindex<LAT, REC>(a, b, 0) >= 0, hindex<LAT, REC>(a, b, 1) >= 0, hindex<LAT, REC>(a, b, 2) >= 0);
}
template <int LAT, bool REC> constexpr bool presU(int a, int cy, int cz)
{
    return syn_present(cy, presT<LAT, REC>(a, 0, cz), presT<LAT, REC>(a, 1, cz), presT<LAT, REC>(a, 2, cz));
}

template <int LAT, bool REC, typename Real, bool U36 = false>
__device__ __forceinline__ void reconstruct_tensor3(const Real (&A)[Basis<LAT, REC>::NH], Real (&f)[Lattice<LAT>::Q])
{
    using L = Lattice<LAT>;
    constexpr bool W = recon_kind<LAT, REC>() == RECON_TENSOR_W;
    auto coef = [&](auto kc) -> Real {
        constexpr int k = decltype(kc)::value;
        if constexpr (k < 0) return Real(0);
        else return A[k];
    };
    Real T[3][3][3]; // [h_x][h_y][c_z + 1]
    static_for<0, 9>([&](auto abk) {
        constexpr int a = decltype(abk)::value / 3, b = decltype(abk)::value % 3;
        constexpr int k0 = hindex<LAT, REC>(a, b, 0), k1 = hindex<LAT, REC>(a, b, 1), k2 = hindex<LAT, REC>(a, b, 2);
        synth_p<W, (k0 >= 0), (k1 >= 0), (k2 >= 0), Real, U36>(coef(std::integral_constant<int, k0>{}),
                                                     coef(std::integral_constant<int, k1>{}),
                                                     coef(std::integral_constant<int, k2>{}), T[a][b][0], T[a][b][1],
                                                     T[a][b][2]);
    });
    Real U[3][3][3]; // [h_x][c_y + 1][c_z + 1]
    static_for<0, 9>([&](auto azk) {
        constexpr int a = decltype(azk)::value / 3, zi = decltype(azk)::value % 3;
        synth_p<W, presT<LAT, REC>(a, 0, zi - 1), presT<LAT, REC>(a, 1, zi - 1), presT<LAT, REC>(a, 2, zi - 1), Real, U36>(T[a][0][zi], T[a][1][zi], T[a][2][zi],
                                                                      U[a][0][zi], U[a][1][zi], U[a][2][zi]);
    });
    Real V[3][3][3]; // [c_x + 1][c_y + 1][c_z + 1]
    static_for<0, 9>([&](auto yzk) {
        constexpr int yi = decltype(yzk)::value / 3, zi = decltype(yzk)::value % 3;
        synth_p<W, presU<LAT, REC>(0, yi - 1, zi - 1), presU<LAT, REC>(1, yi - 1, zi - 1),
                presU<LAT, REC>(2, yi - 1, zi - 1), Real, U36>(
            U[0][yi][zi], U[1][yi][zi], U[2][yi][zi], V[0][yi][zi], V[1][yi][zi], V[2][yi][zi]);
    });
    static_for<0, L::Q>([&](auto ik) {
        constexpr int i = decltype(ik)::value;
        constexpr int xi = L::c[i][0] + 1, yi = L::c[i][1] + 1, zi = L::c[i][2] + 1;
        if constexpr (W) {
            f[i] = V[xi][yi][zi];
        } else {
            constexpr int m36 = int(L::w[i] * 36.0 + 0.5); // 12, 2 or 1 (D3Q19)
            static_assert(m36 == 12 || m36 == 2 || m36 == 1, "TENSOR_U weights");
            if constexpr (m36 == 1) f[i] = V[xi][yi][zi];
            else if constexpr (m36 == 2) f[i] = V[xi][yi][zi] + V[xi][yi][zi];
            else f[i] = Real(12) * V[xi][yi][zi];
        }
    });
}

// Multiply-accumulate by a small compile-time integer.
template <int K, typename Real> __device__ __forceinline__ void acc_int(Real &s, Real v)
{
    if constexpr (K == 1) s += v;
    else if constexpr (K == -1) s -= v;
    else if constexpr (K != 0) s = fma(Real(K), v, s);
}

// Shifted post-collision populations f~*_i = f*_i - w_i (eq 11 / eq 14):
// f~*_i = w_i sum_h He'_h(c_i) A'_h, evaluated for i and opp(i) together from
// the even (E) and odd (O) parts of the basis: f_i = w(E+O), f_opp = w(E-O).
template <int LAT, bool REC, typename Real>
__device__ __forceinline__ void reconstruct(const Real (&A)[Basis<LAT, REC>::NH], Real (&f)[Lattice<LAT>::Q])
{
    using L = Lattice<LAT>;
    using B = Basis<LAT, REC>;
    if constexpr (recon_kind<LAT, REC>() != RECON_PAIR && Lattice<LAT>::D == 3) {
        reconstruct_tensor3<LAT, REC, Real>(A, f);
        return;
    } else if constexpr (tensor_recon<LAT, REC>()) {
        reconstruct_tensor<LAT, Real>(A, f);
        return;
    }
    static_for<0, L::HALF + 1>([&](auto ik) {
        constexpr int i = decltype(ik)::value;
        Real E = Real(0), O = Real(0);
        static_for<0, B::NH>([&](auto hk) {
            constexpr int k = decltype(hk)::value;
            constexpr int h0 = B::h[k][0], h1 = B::h[k][1], h2 = B::h[k][2];
            constexpr int he = he1s(h0, L::c[i][0]) * he1s(h1, L::c[i][1]) * he1s(h2, L::c[i][2]);
            constexpr bool odd = ((h0 == 1) + (h1 == 1) + (h2 == 1)) % 2 == 1;
            if constexpr (odd) acc_int<he>(O, A[k]);
            else acc_int<he>(E, A[k]);
        });
        constexpr Real w = Real(L::w[i]);
        if constexpr (i == 0) {
            f[0] = w * E;
        } else {
            f[i] = w * (E + O);
            f[i + L::HALF] = w * (E - O);
        }
    });
}

// Accumulate one arriving shifted population v with velocity c_k into the
// raw moment accumulators (sum f~, sum c f~, sum c c f~).
template <class L, int k, typename Real> __device__ __forceinline__ void accum(Real (&acc)[L::M], Real v)
{
    constexpr int D = L::D;
    acc[0] += v;
    static_for<0, D>([&](auto ak) {
        constexpr int a = decltype(ak)::value;
        acc_int<L::c[k][a]>(acc[1 + a], v);
        static_for<a, D>([&](auto bk) {
            constexpr int b = decltype(bk)::value;
            acc_int<L::c[k][a] * L::c[k][b]>(acc[pslot<D>(a, b)], v);
        });
    });
}

// ------------------------------------------------------------ factorised accumulation
// Values whose zero-ness is known at compile time (absent lattice directions).
template <bool P, typename Real> struct OV {
    Real v;
};
template <typename Real> struct OV<false, Real> {
};
template <bool A, bool B, typename Real> __device__ __forceinline__ auto ov_add(OV<A, Real> a, OV<B, Real> b)
{
    if constexpr (A && B) return OV<true, Real>{a.v + b.v};
    else if constexpr (A) return a;
    else if constexpr (B) return b;
    else return OV<false, Real>{};
}
template <bool A, bool B, typename Real> __device__ __forceinline__ auto ov_sub(OV<A, Real> a, OV<B, Real> b)
{
    if constexpr (A && B) return OV<true, Real>{a.v - b.v};
    else if constexpr (A) return a;
    else if constexpr (B) return OV<true, Real>{-b.v};
    else return OV<false, Real>{};
}
// acc += sgn * x  (sgn in {-1, 0, +1}, compile time); ASSIGN: acc = sgn * x
// (the first contribution to a fresh accumulator: no zeroing, no add)
template <int SG, bool ASSIGN = false, bool A, typename Real> __device__ __forceinline__ void ov_acc(Real &acc, OV<A, Real> x)
{
    if constexpr (ASSIGN) {
        if constexpr (A && SG == 1) acc = x.v;
        else if constexpr (A && SG == -1) acc = -x.v;
        else acc = Real(0);
    } else {
        if constexpr (A && SG == 1) acc += x.v;
        else if constexpr (A && SG == -1) acc -= x.v;
    }
}
template <class A, class B, class C> struct Tri {
    A r0;
    B r1;
    C r2;
};
// 1D moment sums over c in {-1,0,+1}: r0 = sum g, r1 = sum c g, r2 = sum c^2 g
template <class GM, class G0, class GP> __device__ __forceinline__ auto sums3(GM gm, G0 g0, GP gp)
{
    auto r2 = ov_add(gp, gm);
    auto r1 = ov_sub(gp, gm);
    auto r0 = ov_add(r2, g0);
    return Tri<decltype(r0), decltype(r1), decltype(r2)>{r0, r1, r2};
}

// lattice direction with kernel-axis velocity (ca, cb, cm), or -1
template <class L> constexpr int dir_of(int ca, int cb, int cm)
{
    for (int k = 0; k < L::Q; k++)
        if (Axes<L>::ca(k) == ca && Axes<L>::cb(k) == cb && Axes<L>::cm(k) == cm) return k;
    return -1;
}

// Add the raw moments (sum f, sum c f, sum c c f) of the arrivals G(ia, ib)
// that move by CM along the sweep axis to acc, sum-factorised: sums over c_a
// per row c_b, then over c_b; the sweep component c_m = CM enters as a factor.
// AS: acc is fresh (assigned, not added to).
template <class L, int CM, bool AS, typename Real, class GF>
__device__ __forceinline__ void accum_group(Real (&acc)[L::M], GF &&G)
{
    constexpr int D = L::D;
    using I0 = std::integral_constant<int, 0>;
    using I1 = std::integral_constant<int, 1>;
    using I2 = std::integral_constant<int, 2>;
    // rows: r[ib] over c_a
    auto rm = sums3(G(I0{}, I0{}), G(I1{}, I0{}), G(I2{}, I0{})); // c_b = -1
    auto rz = sums3(G(I0{}, I1{}), G(I1{}, I1{}), G(I2{}, I1{})); // c_b = 0
    auto rp = sums3(G(I0{}, I2{}), G(I1{}, I2{}), G(I2{}, I2{})); // c_b = +1
    // columns over c_b
    auto Sbb = ov_add(rp.r0, rm.r0);                 // sum cb^2 f
    auto Sb = ov_sub(rp.r0, rm.r0);                  // sum cb f
    auto S = ov_add(Sbb, rz.r0);                     // sum f
    auto Sa = ov_add(ov_add(rp.r1, rm.r1), rz.r1);   // sum ca f
    auto Saa = ov_add(ov_add(rp.r2, rm.r2), rz.r2);  // sum ca^2 f
    auto Sab = ov_sub(rp.r1, rm.r1);                 // sum ca cb f
    constexpr int CM2 = CM * CM;
    ov_acc<1, AS>(acc[0], S);
    ov_acc<1, AS>(acc[1], Sa);                       // j_x (A = x)
    if constexpr (D == 3) {
        ov_acc<1, AS>(acc[2], Sb);                   // j_y (B = y)
        ov_acc<CM, AS>(acc[3], S);                   // j_z (C = z)
        ov_acc<1, AS>(acc[pslot<3>(0, 0)], Saa);
        ov_acc<1, AS>(acc[pslot<3>(1, 1)], Sbb);
        ov_acc<CM2, AS>(acc[pslot<3>(2, 2)], S);
        ov_acc<1, AS>(acc[pslot<3>(0, 1)], Sab);
        ov_acc<CM, AS>(acc[pslot<3>(0, 2)], Sa);
        ov_acc<CM, AS>(acc[pslot<3>(1, 2)], Sb);
    } else {                                         // 2D: C = y, no B axis
        ov_acc<CM, AS>(acc[2], S);
        ov_acc<1, AS>(acc[pslot<2>(0, 0)], Saa);
        ov_acc<CM2, AS>(acc[pslot<2>(1, 1)], S);
        ov_acc<CM, AS>(acc[pslot<2>(0, 1)], Sa);
    }
}

// ------------------------------------------------------------ cold paths (out of line)
// Kept out of the fused kernel body so that the hot loop stays small enough
// for the instruction cache; executed only by threads on walls / open faces.
template <typename Real, int M> struct RVec {
    Real v[M];
};

__device__ __forceinline__ double rcp_nr(double x)
{
    // branch-free reciprocal: hardware approximation + 3 Newton steps (to ~1 ulp)
    double r;
    asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
    double e = fma(-x, r, 1.0);
    r = fma(r, e, r);
    e = fma(-x, r, 1.0);
    r = fma(r, e, r);
    e = fma(-x, r, 1.0);
    return fma(r, e, r);
}
__device__ __forceinline__ float rcp_nr(float x)
{
    float r;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
    const float e = fmaf(-x, r, 1.0f);
    return fmaf(r, e, r);
}

// Halfway bounce-back (push form at the emitting node, R12) with the moving-wall
// term (R13): the raw-moment increment of the node's own layer.  fl = this
// thread's slot in the exchange plane (stride NT), holding the movers that
// went through shared memory (SHFL: only those with c_b != 0); the others are
// read from fown; wt weights arrivals on an open face (R14).
// NT: exchange-plane slot stride (0: all of fown is valid); UPOFF: extra offset of the c_b = +1 movers'
// own position (cluster layout: their slot rows start at row -1)
template <int LAT, typename Real, int NT, bool SHFL, int UPOFF = 0>
__device__ __forceinline__ RVec<Real, Lattice<LAT>::M> bounce_back(const Real *fl, const Real (&fown)[Lattice<LAT>::Q],
                                                              int bbA, int bbB, int bbC, Real rho_own,
                                                              const StepArgs *p, int nx_in, int ny_in, bool open)
{
    using L = Lattice<LAT>;
    using X = Axes<L>;
    RVec<Real, L::M> d;
#pragma unroll
    for (int q = 0; q < L::M; q++) d.v[q] = Real(0);
    static_for<0, L::Q>([&](auto kk) {
        constexpr int k = decltype(kk)::value;
        constexpr int ca = X::ca(k), cb = X::cb(k), cm = X::cm(k);
        const bool xA = (ca != 0) && (ca == bbA);
        const bool xB = (cb != 0) && (cb == bbB);
        const bool xC = (cm != 0) && (cm == bbC);
        if (xA || xB || xC) {
            Real v;
            if constexpr (NT == 0) v = fown[k]; // every population passed in registers
            else if constexpr (SHFL && X::bmover(k)) v = fl[X::bslot(k) * NT + (cb > 0 ? UPOFF : 0)];
            else if constexpr (!SHFL && X::moving(k)) v = fl[X::slot(k) * NT];
            else v = fown[k];
            constexpr int kx = L::c[k][0], ky = L::c[k][1], kz = L::c[k][2];
            constexpr double wk6 = 6.0 * L::w[k];
            double cuw = 0.0;
            auto lid = [&](int face) {
                if (p->kind[face] == BC_MOVING) cuw += kx * p->uw[face][0] + ky * p->uw[face][1] + kz * p->uw[face][2];
            };
            if (xA) lid(ca < 0 ? 0 : 1);
            if (xB) lid(cb < 0 ? 2 : 3);
            if (xC) lid(cm < 0 ? 4 : 5);
            v = fma(-(Real(wk6) * rho_own), Real(cuw), v); // explicit: same rounding in every instance
            constexpr int ko = X::opp(k);
            if (open) {
                constexpr int ox = L::c[ko][0], oy = L::c[ko][1];
                const int cn = ox * nx_in + oy * ny_in;
                v *= cn > 0 ? Real(0) : (cn < 0 ? Real(2) : Real(1));
            }
            accum<L, ko>(d.v, v);
        }
    });
    return d;
}

// Regularized open face (R14) finalisation from the weighted raw sums s:
//   velocity face: rho = S0 / (1 - u.n);  pressure face: u.n = 1 - S0 / rho, u_t = 0
//   Pi = SPi - 6 rho sum_{c.n<0} w H (c.u)   (closed form of the f^neq bounce-back rebuild)
template <int LAT, typename Real>
__device__ __forceinline__ RVec<Real, Lattice<LAT>::M> finalize_open(RVec<Real, Lattice<LAT>::M> s, int openF, int nx_in,
                                                                int ny_in, int cg, int a, int b, int nA, int nB,
                                                                const StepArgs *p)
{
    using L = Lattice<LAT>;
    constexpr int D = L::D, Q = L::Q, M = L::M;
    RVec<Real, M> out;
    const Real S0 = s.v[0];
    Real u[3] = {Real(0), Real(0), Real(0)};
    Real drho;
    if (p->kind[openF] == BC_VELOCITY) {
        const double *prof = p->open_prof[openF];
        if (prof) {
            const long long fi = (openF < 2) ? ((long long)cg * nB + b) : ((long long)cg * nA + a);
            for (int q = 0; q < D; q++) u[q] = Real(prof[fi * D + q]);
        } else {
            for (int q = 0; q < D; q++) u[q] = Real(p->open_u[openF][q]);
        }
        const Real un = u[0] * Real(nx_in) + u[1] * Real(ny_in);
        drho = (S0 + un) / (Real(1) - un);
    } else {
        drho = Real(p->open_drho[openF]);
        const Real rho = Real(1) + drho;
        const Real un = (drho - S0) / rho;
        u[0] = un * Real(nx_in);
        u[1] = un * Real(ny_in);
    }
    const Real rho = Real(1) + drho;
    out.v[0] = drho;
    for (int q = 0; q < D; q++) out.v[1 + q] = u[q];
    Real corr[M];
#pragma unroll
    for (int q = 0; q < M; q++) corr[q] = Real(0);
    static_for<0, Q>([&](auto kk) {
        constexpr int k = decltype(kk)::value;
        constexpr int kx = L::c[k][0], ky = L::c[k][1], kz = L::c[k][2];
        constexpr Real wk = Real(L::w[k]);
        const int cn = kx * nx_in + ky * ny_in;
        if (cn < 0) {
            Real cu = Real(kx) * u[0] + Real(ky) * u[1];
            if constexpr (D == 3) cu += Real(kz) * u[2];
            const Real t = wk * cu;
            static_for<0, D>([&](auto qk) {
                constexpr int q = decltype(qk)::value;
                static_for<q, D>([&](auto rk) {
                    constexpr int r = decltype(rk)::value;
                    constexpr Real H = Real(L::c[k][q] * L::c[k][r]) - ((q == r) ? Real(1.0 / 3.0) : Real(0));
                    corr[pslot<D>(q, r)] = fma(H, t, corr[pslot<D>(q, r)]);
                });
            });
        }
    });
#pragma unroll
    for (int q = 0; q < D; q++)
#pragma unroll
        for (int r = q; r < D; r++)
            out.v[pslot<D>(q, r)] = fma(Real(-6) * rho, corr[pslot<D>(q, r)],
                                        (q == r) ? fma(S0, Real(-1.0 / 3.0), s.v[pslot<D>(q, r)]) : s.v[pslot<D>(q, r)]);
    return out;
}

// ------------------------------------------------------------ step kernel
// Accumulator scheme of the sweep (see the kernel): two sets with alternating
// roles, except D3Q27 recursive, whose body unrolled twice spills registers
template <int LAT, bool REC> struct Sweep {
    static constexpr bool two_set = !(LAT == LAT_D3Q27 && REC);
    // a second, boundary-free body for interior CTAs (2D; the 3D bodies are
    // large enough that two of them compete for the instruction cache)
#if defined(MRLBM_NO_FAST_PATH)
    static constexpr bool fast_path = false;
#elif defined(MRLBM_FAST_PATH_3D)
    static constexpr bool fast_path = true;
#else
    static constexpr bool fast_path = LAT == LAT_D2Q9;
#endif
};

// exchange-plane slot of population k, or -1 if it does not go through shared
// memory (SHFL: only the c_b != 0 movers do; the others are shuffled or stay)
template <class L, bool SHFL> constexpr int xslot_of(int k)
{
    if (SHFL) return Axes<L>::bmover(k) ? Axes<L>::bslot(k) : -1;
    return Axes<L>::moving(k) ? Axes<L>::slot(k) : -1;
}

// exchange-plane row of window row r for mover k (cluster layout: the slots of
// the c_b = +1 movers start at row -1, those of the c_b = -1 movers end at row TB)
template <class L, int CL, int k> __device__ __forceinline__ int xrow(int r)
{
    return r + ((CL > 1 && Axes<L>::cb(k) > 0) ? 1 : 0);
}

template <int LAT, typename Real, int TA, int TB, int S, int CL = 1> struct StepSmem {
    using L = Lattice<LAT>;
    static constexpr int NT = TA * TB;
    // cluster of CL CTAs stacked along B (3D): each exchange-plane slot has one
    // extra row -- row -1 for the c_b = +1 movers, row TB for the c_b = -1
    // movers -- that the neighbouring CTA of the cluster fills through DSMEM
    static constexpr int RS = (CL > 1) ? (TB + 1) * TA : NT; // elements per slot
    // 3D tiles one warp wide: populations moving only along A are exchanged
    // with warp shuffles, only the c_b != 0 movers go through shared memory
    static constexpr bool SHFL = L::D == 3 && TA == 32;
    static constexpr int NX = SHFL ? Axes<L>::NBMOVE : Axes<L>::NMOVE; // movers in the exchange plane
    // TMA box rows must start on a 16-byte boundary: the box starts at the
    // window origin rounded down to AL elements and is BW elements wide.
    static constexpr int AL = 16 / int(sizeof(Real));
    static constexpr int BW = (TA + AL - 1 + AL - 1) / AL * AL;
    static constexpr size_t box_elems = size_t(L::M) * TB * BW;
    static constexpr size_t stage_elems = (box_elems * sizeof(Real) + 127) / 128 * 128 / sizeof(Real);
    static constexpr size_t F_elems = size_t(NX) * RS; // one exchange plane
    // two exchange planes (alternating layers) -> one __syncthreads per layer
    static constexpr size_t bytes = (S * stage_elems + 2 * F_elems) * sizeof(Real) + S * sizeof(uint64_t) + 128;
};

// PUSH: the P2P-transport instance for a rank's boundary layers (peer stores);
// the plain instance carries none of that code
// CL > 1 (3D): launched in clusters of CL CTAs along B (grid.y); the CTAs of a
// cluster stack their windows and only the cluster's outermost rows are halo
// rows (owned rows per cluster CL*TB - 2 instead of CL*(TB - 2)); movers that
// cross an inner CTA boundary are stored straight into the neighbour CTA's
// exchange plane (DSMEM) and the per-layer barrier is cluster-wide.
template <int LAT, bool REC, typename Real, int TA, int TB, int S, int MINB, bool PUSH = false, int CL = 1>
__global__ void __launch_bounds__(TA *TB, MINB) mrlbm_step_kernel(const __grid_constant__ CUtensorMap tmap,
                                                            const StepArgs p)
{
    using L = Lattice<LAT>;
    using X = Axes<L>;
    constexpr int D = L::D, Q = L::Q, M = L::M;
    constexpr int NT = TA * TB;
    using SM = StepSmem<LAT, Real, TA, TB, S, CL>;
    constexpr bool SHFL = SM::SHFL;
    static_assert(CL == 1 || (D == 3 && SHFL), "clusters: 3D one-warp-wide tiles only");
    constexpr int RS = SM::RS;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    Real *stage = reinterpret_cast<Real *>(smem_raw);
    Real *Fs = stage + S * SM::stage_elems;
    uint64_t *full = reinterpret_cast<uint64_t *>(Fs + 2 * SM::F_elems);

    const int tid = threadIdx.x;
    const int tx = tid % TA, ty = tid / TA;
    // grid: x = tile along A, y = tile along B (CL consecutive CTAs = one
    // cluster), z = sweep segment
    // Launch order (3D, no clusters): consecutive CTAs walk groups of rastG
    // B-neighbours, group by group along A, so that the CTAs sharing a halo row
    // (B) or halo columns (A) run close together in time and their shared
    // box rows are L2 hits rather than second DRAM reads.
    int tA = blockIdx.x, tBi = blockIdx.y;
    if (D == 3 && CL == 1 && p.rastG > 0) {
        const int L = blockIdx.x;
        const int span = p.rastG * p.tilesA;
        const int grp = L / span;
        const int w = L - grp * span;
        const int g0 = grp * p.rastG;
        const int gsz = min(p.rastG, p.tilesB - g0);
        tA = w / gsz;
        tBi = g0 + (w - tA * gsz);
    }
    const int kcl = (CL > 1) ? int(cluster_ctarank()) : 0;
    const int a0 = tA * (TA - 2) - 1;
    const int b0 = (D == 3) ? (tBi / CL) * (CL * TB - 2) - 1 + kcl * TB : 0;
    const int a = a0 + tx, b = b0 + ty;
    const int nA = p.nA, nB = p.nB, nC = p.nC;
    // window rows owned by this CTA: all but the cluster's outermost rows
    const int row_lo = (D == 3 && kcl == 0) ? 1 : 0;
    const int row_hi = (D == 3 && kcl == CL - 1) ? TB - 2 : TB - 1;

    const bool second = (int)blockIdx.z >= p.nseg1;
    const int c0 = second ? p.c2_begin + ((int)blockIdx.z - p.nseg1) * p.seg_len : p.c_begin + blockIdx.z * p.seg_len;
    const int c1 = min(c0 + p.seg_len, second ? p.c2_end : p.c_end);
    if (c0 >= c1) return;
    const int boxA = ((a0 + p.padA) / SM::AL) * SM::AL; // aligned TMA box origin (a0 + padA >= 0)
    const int offA = a0 + p.padA - boxA;                  // window column 0 inside the box
    const int cfirst = (c0 > 0 || p.lo_nb) ? c0 - 1 : c0;
    const int clast = (c1 < nC || p.hi_nb) ? c1 : c1 - 1;
    const int nl = clast - cfirst + 1;

    // Fast CTAs: the whole window lies inside the domain, no owner sits on a
    // domain face or a periodic edge, and the segment holds neither the first
    // nor the last layer -- no wall, open face, ghost copy or peer push can
    // occur, so that body is compiled without any of their tests (most CTAs)
    const bool fast_cta = Sweep<LAT, REC>::fast_path && a0 >= 0 && a0 + TA <= nA &&
                          (D == 2 || (b0 >= 0 && b0 + TB <= nB)) && c0 > 0 && c1 < nC;
    auto run = [&](auto fast_tag) {
    constexpr bool FAST = decltype(fast_tag)::value;

    // ---- per-thread roles
    const bool perA = p.kind[0] == BC_PERIODIC, perB = p.kind[2] == BC_PERIODIC;
    const bool inA = a >= 0 && a < nA, inB = b >= 0 && b < nB;
    // Every window position is computed, node or not: positions that hold no
    // node (pads outside a non-periodic face, TMA out-of-bounds boxes) read
    // all-zero moments (the buffers are zeroed at creation and only nodes and
    // periodic ghosts are ever stored), and zero shifted moments (rho - 1 = 0,
    // u = 0, Pi = 0) collide and reconstruct to exactly zero shifted
    // populations -- so they publish zeros and the pulls need no predicate.
    const bool interior = tx >= 1 && tx < TA - 1 && ty >= row_lo && ty <= row_hi;
    const bool owner = FAST ? interior : (interior && inA && inB);
    // SHFL: every lane of an interior row runs the streaming code (a warp is one
    // row, so the shuffles see all 32 lanes); only owners store
    const bool stream_lane = SHFL ? (ty >= row_lo && ty <= row_hi) : owner;
    // open faces in this CTA's window (CTA-uniform, so that the weighted and the
    // plain streaming bodies never diverge inside a warp)
    // (a superset: the weighted body is also correct where no node is open)
    const bool cta_open = !FAST && ((p.kind[0] >= BC_VELOCITY && a0 < 0) || (p.kind[1] >= BC_VELOCITY && a0 + TA - 1 >= nA - 1) ||
                                    (D == 3 && ((p.kind[2] >= BC_VELOCITY && b0 <= 0) ||
                                                (p.kind[3] >= BC_VELOCITY && b0 + TB - 1 >= nB - 1))));
    // ghost shift of an owner on a periodic edge: a = 0 -> column nA, a = nA-1 -> column -1
    const int gA = (FAST || !perA) ? 0 : (a == 0 ? nA : (a == nA - 1 ? -nA : 0));
    const int gB = (D == 2 || !perB) ? 0 : (b == 0 ? nB : (b == nB - 1 ? -nB : 0));
    // pull-source availability along A/B: source at a-1 (c_a = +1), a+1 (c_a = -1)
    // walls touching this node in-plane (-1 lower face, +1 upper face)
    auto is_wall = [](int k) { return k == BC_WALL || k == BC_MOVING; };
    const int bbA = FAST ? 0 : ((a == 0 && is_wall(p.kind[0])) ? -1 : ((a == nA - 1 && is_wall(p.kind[1])) ? 1 : 0));
    const int bbB = (D == 2) ? 0 : ((b == 0 && is_wall(p.kind[2])) ? -1 : ((b == nB - 1 && is_wall(p.kind[3])) ? 1 : 0));
    // open face of this node (index 0..3 into open_*), inward normal (physical x / y)
    int openF = -1, nx_in = 0, ny_in = 0;
    if (!FAST && owner) {
        if (a == 0 && p.kind[0] >= BC_VELOCITY) { openF = 0; nx_in = 1; }
        else if (a == nA - 1 && p.kind[1] >= BC_VELOCITY) { openF = 1; nx_in = -1; }
        else if (D == 3 && b == 0 && p.kind[2] >= BC_VELOCITY) { openF = 2; ny_in = 1; }
        else if (D == 3 && b == nB - 1 && p.kind[3] >= BC_VELOCITY) { openF = 3; ny_in = -1; }
    }

    const Real *src = reinterpret_cast<const Real *>(p.src);
    Real *dst = reinterpret_cast<Real *>(p.dst);
    const Real omega = Real(p.omega);
    auto plane_of = [&](int c) -> int { return p.wrapC ? ((c % nC + nC) % nC) + 1 : c + 1; };

    // ---- TMA ring prologue
    if (tid == 0) {
        prefetch_tmap(&tmap);
#pragma unroll
        for (int s = 0; s < S; s++) mbar_init(&full[s], 1);
        fence_barrier_init();
    }
    // clusters: every CTA of the cluster is running (its shared memory may
    // receive DSMEM stores) once this barrier completes
    if constexpr (CL > 1) cluster_sync_all();
    else __syncthreads();
    constexpr uint32_t stage_bytes = uint32_t(SM::box_elems * sizeof(Real)); // bytes one TMA box delivers
    if (tid == 0) {
        for (int s = 0; s < S && s < nl; s++) {
            mbar_expect_tx(&full[s], stage_bytes);
            tma_load_4d(stage + s * SM::stage_elems, &tmap, &full[s], boxA, b0 + p.padB, 0, plane_of(cfirst + s));
        }
    }

    // Two accumulator sets suffice for the three layers an arrival can reach
    // (c-1, c, c+1): layer c-1 is completed and stored by the c_m = -1 group
    // before anything is added to layer c+1, whose sums then reuse its
    // registers.  The roles of the two sets alternate from layer to layer
    // (the sweep is unrolled by two), so no accumulator is ever moved.
    Real accA[M], accB[M], accC[M];
#pragma unroll
    for (int q = 0; q < M; q++) {
        accA[q] = Real(0);
        accB[q] = Real(0);
        accC[q] = Real(0);
    }

    // ---- finalize the completed layer and store it (eqs 1-3; open faces R14)
    Real *const dst_node = dst + (long long)b * p.pitch + a; // this thread's node in plane 0
    auto finalize_store = [&](const Real (&s)[M], int c) {
        Real out[M];
        const Real S0 = s[0];
        if (openF < 0) {
            const Real inv = rcp_nr(Real(1) + S0);
            out[0] = S0;
#pragma unroll
            for (int q = 0; q < D; q++) out[1 + q] = s[1 + q] * inv;
#pragma unroll
            for (int q = 0; q < D; q++)
#pragma unroll
                for (int r = q; r < D; r++)
                    out[pslot<D>(q, r)] = (q == r) ? fma(S0, Real(-1.0 / 3.0), s[pslot<D>(q, r)]) : s[pslot<D>(q, r)];
        } else {
            RVec<Real, M> sv;
#pragma unroll
            for (int q = 0; q < M; q++) sv.v[q] = s[q];
            const RVec<Real, M> ov = finalize_open<LAT, Real>(sv, openF, nx_in, ny_in, c + p.c_offset, a, b, nA, nB, &p);
#pragma unroll
            for (int q = 0; q < M; q++) out[q] = ov.v[q];
        }
        if (!owner) return;
        Real *o = dst_node + (long long)(c + 1) * p.pstride;
        auto store_plane = [&](Real *o) {
            const int ms = int(p.mstride); // < 2^31 elements per moment plane (32-bit offsets)
#pragma unroll
            for (int q = 0; q < M; q++) o[q * ms] = out[q];
            // periodic ghost copies of edge nodes (also the corner ghosts)
            if (gA | gB) {
                auto put = [&](int da, int db) {
                    Real *g = o + (long long)db * p.pitch + da;
#pragma unroll
                    for (int q = 0; q < M; q++) g[q * ms] = out[q];
                };
                if (gA) put(gA, 0);
                if (gB) put(0, gB);
                if (gA && gB) put(gA, gB);
            }
        };
        store_plane(o);
        // P2P halo push: the slab's first / last layer also goes straight into
        // the neighbour's ghost plane (peer memory), same in-plane layout
        if constexpr (PUSH && !FAST) {
            void *peer = (c == 0) ? p.peer_lo : ((c == nC - 1) ? p.peer_hi : nullptr);
            if (peer) {
                store_plane(reinterpret_cast<Real *>(peer) + (long long)b * p.pitch + a);
                __threadfence_system();
            }
        }
    };

    // one layer of the sweep: on entry X holds layer c-1 and Y layer c; on
    // exit Y holds layer c and Z layer c+1.  Z is X (ALIAS, two-set scheme)
    // or a third, zeroed set (rotation scheme)
    auto layer = [&](const int it, Real (&X)[M], Real (&Y)[M], Real (&Z)[M]) {
        const int c = cfirst + it;
        const int s = it % S;
        mbar_wait(&full[s], (it / S) & 1);

        Real m[M];
        {
            const Real *st = stage + s * SM::stage_elems + ty * SM::BW + tx + offA;
#pragma unroll
            for (int q = 0; q < M; q++) m[q] = st[q * (TB * SM::BW)];
        }
        // ---- collide + reconstruct (eqs 10-14) and publish the in-plane movers
        // into exchange plane it & 1 (positions without a node publish zeros,
        // so pulls need no validity predicate; arrivals into layers that do not
        // exist land in accumulators that are never stored)
        Real *Fl = Fs + (it & 1) * SM::F_elems;
        Real fown[Q]; // only the non-moving entries are used after the barrier
        const Real rho_own = Real(1) + m[0];
        {
            Real A[Basis<LAT, REC>::NH];
            if constexpr (LAT == LAT_D3Q19) {
                // regrouped collision, Hermite scales applied per axis by the synthesis
                collide_u36<REC, Real>(m, omega, A);
                reconstruct_tensor3<LAT, REC, Real, true>(A, fown);
            } else {
                collide_coeffs<LAT, REC, Real>(m, omega, A);
                reconstruct<LAT, REC, Real>(A, fown);
            }
        }
        static_for<0, Q>([&](auto kk) {
            constexpr int k = decltype(kk)::value;
            constexpr int xs = xslot_of<L, SM::SHFL>(k);
            if constexpr (xs >= 0) Fl[xs * RS + xrow<L, CL, k>(ty) * TA + tx] = fown[k];
        });
        if constexpr (CL > 1) {
            // movers leaving through an inner cluster boundary go straight into
            // the neighbour CTA's exchange plane: row 0's c_b = -1 movers become
            // row TB of CTA kcl - 1, row TB-1's c_b = +1 movers row -1 of kcl + 1
            if (ty == 0 && kcl > 0) {
                const uint32_t base = mapa_shared(smem_u32(Fl), uint32_t(kcl - 1));
                static_for<0, Q>([&](auto kk) {
                    constexpr int k = decltype(kk)::value;
                    if constexpr (X::cb(k) < 0)
                        st_cluster(base + uint32_t((X::bslot(k) * RS + TB * TA + tx) * sizeof(Real)), fown[k]);
                });
            }
            if (ty == TB - 1 && kcl < CL - 1) {
                const uint32_t base = mapa_shared(smem_u32(Fl), uint32_t(kcl + 1));
                static_for<0, Q>([&](auto kk) {
                    constexpr int k = decltype(kk)::value;
                    if constexpr (X::cb(k) > 0)
                        st_cluster(base + uint32_t((X::bslot(k) * RS + tx) * sizeof(Real)), fown[k]);
                });
            }
        }
        // one barrier per layer (cluster-wide with CL > 1): the other exchange
        // plane was last read before this barrier, and every thread has read
        // stage s
        if constexpr (CL > 1) cluster_sync_all();
        else __syncthreads();
        if (tid == 0 && it + S < nl) {
            mbar_expect_tx(&full[s], stage_bytes);
            tma_load_4d(stage + s * SM::stage_elems, &tmap, &full[s], boxA, b0 + p.padB, 0, plane_of(c + S));
        }

        if (stream_lane) {
            const int bbC = FAST ? 0 : ((c == 0 && !p.lo_nb) ? -1 : ((c == nC - 1 && !p.hi_nb) ? 1 : 0));
            auto body = [&](auto open_tag) {
                constexpr bool OPEN = decltype(open_tag)::value;
                auto wt = [&](int kx, int ky) -> Real {
                    const int cn = kx * nx_in + ky * ny_in;
                    return cn > 0 ? Real(0) : (cn < 0 ? Real(2) : Real(1));
                };
                // streaming (eq 7), pull form across the tile; C-moves stay in
                // registers.  Arrivals for layer c-1 first, so that layer c-1
                // is finalized and its accumulators freed before layers c, c+1
                // are accumulated (lower register pressure).
                auto pull = [&](auto cm_tag) {
                    constexpr int CM = decltype(cm_tag)::value;
                    auto G = [&](auto iac, auto ibc) {
                        constexpr int ca = decltype(iac)::value - 1, cb = decltype(ibc)::value - 1;
                        constexpr int k = dir_of<L>(ca, cb, CM);
                        if constexpr (k < 0) {
                            return OV<false, Real>{};
                        } else {
                            Real v;
                            constexpr int xs = xslot_of<L, SM::SHFL>(k);
                            if constexpr (xs >= 0) v = Fl[xs * RS + xrow<L, CL, k>(ty - cb) * TA + (tx - ca)];
                            else if constexpr (ca != 0) v = __shfl_sync(0xffffffffu, fown[k], tx - ca);
                            else v = fown[k];
                            if constexpr (OPEN) {
                                constexpr int kx = L::c[k][0], ky = L::c[k][1];
                                v *= wt(kx, ky);
                            }
                            return OV<true, Real>{v};
                        }
                    };
                    // the c_m = +1 group is the first contribution to layer c+1
                    accum_group<L, CM, (CM > 0), Real>(CM < 0 ? X : (CM == 0 ? Y : Z), G);
                };
                pull(std::integral_constant<int, -1>{});
                if (c - 1 >= c0 && c - 1 < c1) finalize_store(X, c - 1);
                pull(std::integral_constant<int, 0>{});
                pull(std::integral_constant<int, 1>{}); // assigns Z (= X in the two-set scheme)
                // halfway bounce-back at walls (R12, R13), out of line
                if (bbA | bbB | bbC) {
                    const RVec<Real, M> d = bounce_back<LAT, Real, RS, SM::SHFL, (CL > 1 ? TA : 0)>(Fl + tid, fown, bbA, bbB, bbC, rho_own, &p,
                                                                             nx_in, ny_in, OPEN);
#pragma unroll
                    for (int q = 0; q < M; q++) Y[q] += d.v[q];
                }
            };
            if (SM::SHFL ? cta_open : openF >= 0) body(std::true_type{});
            else body(std::false_type{});
        }
    };
    if constexpr (Sweep<LAT, REC>::two_set && CL == 1 && D == 3 && MRLBM_ROTATE_SCALAR) {
        // Rotated sweep: the barrier closes each iteration, and the block between
        // two barriers holds the pulls of layer it AND the collision +
        // reconstruction of layer it + 1, which are independent -- the compiler
        // interleaves the two dependency chains (latency hiding within a warp).
        // Plane it & 1 is read by consume(it) and next written by produce(it + 2),
        // two barriers later; stage it % S is read by produce(it) before the
        // barrier that precedes its refill.
        Real fA[Q], fB[Q];
        Real rA = Real(1), rB = Real(1);
        auto produce = [&](const int it, Real (&fown)[Q], Real &rho_own) __attribute__((always_inline)) {
            const int s = it % S;
            mbar_wait(&full[s], (it / S) & 1);
            Real m[M];
            const Real *st = stage + s * SM::stage_elems + ty * SM::BW + tx + offA;
#pragma unroll
            for (int q = 0; q < M; q++) m[q] = st[q * (TB * SM::BW)];
            rho_own = Real(1) + m[0];
            Real A[Basis<LAT, REC>::NH];
            if constexpr (LAT == LAT_D3Q19) {
                collide_u36<REC, Real>(m, omega, A);
                reconstruct_tensor3<LAT, REC, Real, true>(A, fown);
            } else {
                collide_coeffs<LAT, REC, Real>(m, omega, A);
                reconstruct<LAT, REC, Real>(A, fown);
            }
            Real *Fl = Fs + (it & 1) * SM::F_elems;
            static_for<0, Q>([&](auto kk) {
                constexpr int k = decltype(kk)::value;
                constexpr int xs = xslot_of<L, SM::SHFL>(k);
                if constexpr (xs >= 0) Fl[xs * RS + ty * TA + tx] = fown[k];
            });
        };
        auto sync_refill = [&](const int it) __attribute__((always_inline)) {
            __syncthreads();
            if (tid == 0 && it + S < nl) {
                const int s = it % S;
                mbar_expect_tx(&full[s], stage_bytes);
                tma_load_4d(stage + s * SM::stage_elems, &tmap, &full[s], boxA, b0 + p.padB, 0, plane_of(cfirst + it + S));
            }
        };
        auto consume = [&](const int it, Real (&X)[M], Real (&Y)[M], Real (&Z)[M], const Real (&fown)[Q],
                           const Real rho_own) __attribute__((always_inline)) {
            if (!stream_lane) return;
            const int c = cfirst + it;
            const Real *Fl = Fs + (it & 1) * SM::F_elems;
            const int bbC = FAST ? 0 : ((c == 0 && !p.lo_nb) ? -1 : ((c == nC - 1 && !p.hi_nb) ? 1 : 0));
            auto body = [&](auto open_tag) __attribute__((always_inline)) {
                constexpr bool OPEN = decltype(open_tag)::value;
                auto wt = [&](int kx, int ky) -> Real {
                    const int cn = kx * nx_in + ky * ny_in;
                    return cn > 0 ? Real(0) : (cn < 0 ? Real(2) : Real(1));
                };
                auto pull = [&](auto cm_tag) __attribute__((always_inline)) {
                    constexpr int CM = decltype(cm_tag)::value;
                    auto G = [&](auto iac, auto ibc) {
                        constexpr int ca = decltype(iac)::value - 1, cb = decltype(ibc)::value - 1;
                        constexpr int k = dir_of<L>(ca, cb, CM);
                        if constexpr (k < 0) {
                            return OV<false, Real>{};
                        } else {
                            Real v;
                            constexpr int xs = xslot_of<L, SM::SHFL>(k);
                            if constexpr (xs >= 0) v = Fl[xs * RS + (ty - cb) * TA + (tx - ca)];
                            else if constexpr (ca != 0) v = __shfl_sync(0xffffffffu, fown[k], tx - ca);
                            else v = fown[k];
                            if constexpr (OPEN) {
                                constexpr int kx = L::c[k][0], ky = L::c[k][1];
                                v *= wt(kx, ky);
                            }
                            return OV<true, Real>{v};
                        }
                    };
                    accum_group<L, CM, (CM > 0), Real>(CM < 0 ? X : (CM == 0 ? Y : Z), G);
                };
                pull(std::integral_constant<int, -1>{});
                if (c - 1 >= c0 && c - 1 < c1) finalize_store(X, c - 1);
                pull(std::integral_constant<int, 0>{});
                pull(std::integral_constant<int, 1>{});
                if (bbA | bbB | bbC) {
                    const RVec<Real, M> d = bounce_back<LAT, Real, RS, SM::SHFL, 0>(Fl + tid, fown, bbA, bbB, bbC, rho_own, &p,
                                                                                nx_in, ny_in, OPEN);
#pragma unroll
                    for (int q = 0; q < M; q++) Y[q] += d.v[q];
                }
            };
            if (SM::SHFL ? cta_open : openF >= 0) body(std::true_type{});
            else body(std::false_type{});
        };
        produce(0, fA, rA);
        sync_refill(0);
        for (int it = 0; it < nl; it += 2) {
            if (it + 1 < nl) produce(it + 1, fB, rB);
            consume(it, accA, accB, accA, fA, rA);
            if (it + 1 < nl) {
                sync_refill(it + 1);
                if (it + 2 < nl) produce(it + 2, fA, rA);
                consume(it + 1, accB, accA, accB, fB, rB);
                if (it + 2 < nl) sync_refill(it + 2);
            }
        }
        if (owner && clast == c1 - 1) {
            if (nl & 1) finalize_store(accB, c1 - 1);
            else finalize_store(accA, c1 - 1);
        }
    } else if constexpr (Sweep<LAT, REC>::two_set) {
        for (int it = 0; it < nl; it += 2) {
            layer(it, accA, accB, accA);
            if (it + 1 < nl) layer(it + 1, accB, accA, accB);
        }
        // the last layer of the segment, when no halo layer follows it, is
        // complete after the sweep: it is the Y of the last layer call
        if (owner && clast == c1 - 1) {
            if (nl & 1) finalize_store(accB, c1 - 1);
            else finalize_store(accA, c1 - 1);
        }
    } else {
        // D3Q27 recursive: the body unrolled twice no longer fits the register
        // file (local-memory spills), so one body and three rotating sets
        for (int it = 0; it < nl; it++) {
            layer(it, accA, accB, accC);
#pragma unroll
            for (int q = 0; q < M; q++) { // accC is assigned by the next layer's c_m = +1 group
                accA[q] = accB[q];
                accB[q] = accC[q];
            }
        }
        if (owner && clast == c1 - 1) finalize_store(accA, c1 - 1);
    }
    };
    if (fast_cta) run(std::true_type{});
    else run(std::false_type{});
}

// ------------------------------------------------------------ finite-difference open faces
// Latt et al. [6] "FD" inlet / outlet (the paper's proxy apps; R20),
// run after the fused step on the new state: the fused kernel has set rho and
// u of the face nodes by the regularized rule (R14); this pass replaces their
// stress by the Chapman-Enskog value of the new velocity field,
//   Pi = rho u u - rho tau c_s^2 (d_a u_b + d_b u_a),
// second-order differences: one-sided along the face normal and at the face's
// edges, central elsewhere (wrapped on periodic axes).  Reads u, writes Pi of
// face nodes only (plus their periodic ghost copies), so there is no hazard.
struct FdArgs {
    void *buf;          // node (0,0) of plane 0 of the state to update
    int nA, nB, nC, pitch;
    long long mstride, pstride;
    int face;           // kernel face 0 A-, 1 A+, 2 B-, 3 B+
    int per[3];         // periodic kernel axes A, B, C
    double tau;
};

template <int LAT, typename Real> __global__ void fd_face_kernel(FdArgs g)
{
    using L = Lattice<LAT>;
    constexpr int D = L::D;
    Real *buf = reinterpret_cast<Real *>(g.buf);
    const int ax = g.face / 2;                    // kernel axis of the face normal
    const int n[3] = {g.nA, g.nB, g.nC};
    const long long nodes = (long long)(ax == 0 ? g.nB : g.nA) * g.nC;
    // kernel axis -> physical axis (2D: A = x, C = y; 3D: A = x, B = y, C = z)
    const int phys[3] = {0, 1, D == 3 ? 2 : 1};
    for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < nodes; t += (long long)gridDim.x * blockDim.x) {
        int idx[3];
        idx[2] = (int)(t / (ax == 0 ? g.nB : g.nA));
        const int r = (int)(t % (ax == 0 ? g.nB : g.nA));
        idx[ax] = (g.face % 2 == 0) ? 0 : n[ax] - 1;
        idx[1 - ax] = r;
        auto at = [&](int a, int b, int c) -> const Real * {
            return buf + (long long)(c + 1) * g.pstride + (long long)b * g.pitch + a;
        };
        auto u_at = [&](const int (&q)[3], int comp) -> Real { return at(q[0], q[1], q[2])[(1 + comp) * g.mstride]; };
        Real grad[3][3] = {}; // grad[a][b] = d_a u_b, physical axes
#pragma unroll
        for (int X = 0; X < 3; X++) {
            if (D == 2 && X == 1) continue;
            const int i = idx[X], nx = n[X];
            int q0[3] = {idx[0], idx[1], idx[2]}, q1[3] = {idx[0], idx[1], idx[2]}, q2[3] = {idx[0], idx[1], idx[2]};
            const bool central = g.per[X] || (i > 0 && i < nx - 1);
            if (central) {
                q1[X] = (i + 1) % nx;
                q2[X] = (i - 1 + nx) % nx;
            } else {
                const int s = (i == 0) ? 1 : -1;
                q1[X] = i + s;
                q2[X] = i + 2 * s;
            }
#pragma unroll
            for (int b = 0; b < D; b++) {
                Real d;
                if (central) d = Real(0.5) * (u_at(q1, b) - u_at(q2, b));
                else d = Real(i == 0 ? 0.5 : -0.5) * (Real(-3) * u_at(q0, b) + Real(4) * u_at(q1, b) - u_at(q2, b));
                grad[phys[X]][b] = d;
            }
        }
        Real *node = buf + (long long)(idx[2] + 1) * g.pstride + (long long)idx[1] * g.pitch + idx[0];
        const Real rho = Real(1) + node[0];
        Real u[3] = {Real(0), Real(0), Real(0)};
#pragma unroll
        for (int b = 0; b < D; b++) u[b] = node[(1 + b) * g.mstride];
        const Real k = -rho * Real(g.tau) * Real(1.0 / 3.0);
        // periodic ghost copy of this face node (in-plane axis along the face)
        long long goff = 0;
        if (ax == 0 && D == 3 && g.per[1]) goff = idx[1] == 0 ? (long long)g.nB * g.pitch : (idx[1] == g.nB - 1 ? -(long long)g.nB * g.pitch : 0);
        if (ax == 1 && g.per[0]) goff = idx[0] == 0 ? g.nA : (idx[0] == g.nA - 1 ? -g.nA : 0);
#pragma unroll
        for (int a = 0; a < D; a++)
#pragma unroll
            for (int b = a; b < D; b++) {
                const Real v = fma(k, grad[a][b] + grad[b][a], rho * u[a] * u[b]);
                node[pslot<D>(a, b) * g.mstride] = v;
                if (goff) node[pslot<D>(a, b) * g.mstride + goff] = v;
            }
    }
}

// Prologue push after the state was set from outside: whole planes (pads and
// in-plane ghosts included) into the neighbours' ghost planes.
template <typename Real>
__global__ void p2p_push_planes_kernel(const Real *own_first, const Real *own_last, Real *peer_lo, Real *peer_hi,
                                       long long count)
{
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < count; i += (long long)gridDim.x * blockDim.x) {
        if (peer_lo) peer_lo[i] = own_first[i];
        if (peer_hi) peer_hi[i] = own_last[i];
    }
    __threadfence_system();
}

// ------------------------------------------------------------ side kernels
struct GridArgs {
    int nA, nB, nC, pitch;
    long long mstride, pstride;
    int perA, perB; // periodic in-plane axes: write ghost copies (set_moments)
};

// ABI fp64 [M][nC][nB][nA] (rho, u, Pi) -> internal Real layout (rho - 1).
template <int M, typename Real>
__global__ void set_moments_kernel(const double *__restrict__ in, Real *__restrict__ buf, GridArgs g)
{
    const long long N = (long long)g.nA * g.nB * g.nC;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        const int a = n % g.nA;
        const int b = (n / g.nA) % g.nB;
        const int c = n / ((long long)g.nA * g.nB);
        Real *o = buf + (long long)(c + 1) * g.pstride + (long long)b * g.pitch + a;
        const int gA = !g.perA ? 0 : (a == 0 ? g.nA : (a == g.nA - 1 ? -g.nA : 0));
        const int gB = !g.perB ? 0 : (b == 0 ? g.nB : (b == g.nB - 1 ? -g.nB : 0));
#pragma unroll
        for (int q = 0; q < M; q++) {
            double v = in[q * N + n];
            if (q == 0) v -= 1.0;
            o[q * g.mstride] = Real(v);
            if (gA) o[q * g.mstride + gA] = Real(v);
            if (gB) o[q * g.mstride + (long long)gB * g.pitch] = Real(v);
            if (gA && gB) o[q * g.mstride + (long long)gB * g.pitch + gA] = Real(v);
        }
    }
}

template <int M, typename Real>
__global__ void get_moments_kernel(const Real *__restrict__ buf, double *__restrict__ out, GridArgs g)
{
    const long long N = (long long)g.nA * g.nB * g.nC;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        const int a = n % g.nA;
        const int b = (n / g.nA) % g.nB;
        const int c = n / ((long long)g.nA * g.nB);
        const Real *i = buf + (long long)(c + 1) * g.pstride + (long long)b * g.pitch + a;
#pragma unroll
        for (int q = 0; q < M; q++) {
            double v = double(i[q * g.mstride]);
            if (q == 0) v += 1.0;
            out[q * N + n] = v;
        }
    }
}

// Post-collision populations f* = f~* + w of every node (R17), fp64 [Q][N].
template <int LAT, bool REC, typename Real>
__global__ void populations_kernel(const Real *__restrict__ buf, double *__restrict__ out, GridArgs g, double omega)
{
    using L = Lattice<LAT>;
    const long long N = (long long)g.nA * g.nB * g.nC;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        const int a = n % g.nA;
        const int b = (n / g.nA) % g.nB;
        const int c = n / ((long long)g.nA * g.nB);
        const Real *i = buf + (long long)(c + 1) * g.pstride + (long long)b * g.pitch + a;
        Real m[L::M];
#pragma unroll
        for (int q = 0; q < L::M; q++) m[q] = i[q * g.mstride];
        Real A[Basis<LAT, REC>::NH];
        Real f[L::Q];
        collide_coeffs<LAT, REC, Real>(m, Real(omega), A);
        reconstruct<LAT, REC, Real>(A, f);
        static_for<0, L::Q>([&](auto kk) {
            constexpr int k = decltype(kk)::value;
            constexpr double wk = L::w[k];
            out[k * N + n] = double(f[k]) + wk;
        });
    }
}

template <int M, typename Real>
__global__ void finite_kernel(const Real *__restrict__ buf, GridArgs g, int *flag)
{
    const long long N = (long long)g.nA * g.nB * g.nC;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        const int a = n % g.nA;
        const int b = (n / g.nA) % g.nB;
        const int c = n / ((long long)g.nA * g.nB);
        const Real *i = buf + (long long)(c + 1) * g.pstride + (long long)b * g.pitch + a;
#pragma unroll
        for (int q = 0; q < M; q++)
            if (!isfinite(double(i[q * g.mstride]))) atomicExch(flag, 1);
    }
}

} // namespace mr
