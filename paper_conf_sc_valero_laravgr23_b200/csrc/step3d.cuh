// step3d.cuh -- the 3D fused MR-LBM step with paired populations (round 3).
//
// Same timestep as mrlbm_step_kernel (Alg. 2; eqs 10-14
// collide + reconstruct, eq 7 streaming, eqs 1-3 moments), same TMA ring,
// same tile (one warp = one A-row of a 32 x TB tile, rolling per-layer
// accumulators along the sweep axis C), but every population that moves along
// C travels as a PAIR with its mirror: (f(ca, cb, -1), f(ca, cb, +1)).
//
//  * The sum-factorised synthesis (eq 14, per axis z, y, x) is run on two
//    chains after the z step: the c_z = 0 chain on scalars and the c_z = +-1
//    chain on pairs, so the y and x steps of both signs share instructions.
//  * A pair is one 64-bit (fp32) / 128-bit (fp64) shared-memory store and load.
//  * The pulled c_m = -1 and c_m = +1 groups (they have identical in-plane
//    structure) are summed together, pair by pair; the low half goes to layer
//    c-1, the high half starts layer c+1.
//  * fp32 pairs are Blackwell packed FP32 (FFMA2 / FADD2 / FMUL2, sm_100):
//    one issue slot for two lanes' worth of FMAs, scalar operands broadcast
//    for free.  fp64 pairs are two scalar ops (DFMA has no packed form).
// Rounding: every population and sum is formed by the same operations in
// the same order as in the scalar kernel's factorisation, so the pair form
// changes which instruction computes a value, not the value's accuracy class.
#pragma once
#include "mrlbm_kernels.cuh"

namespace mr {

// inline every lambda of the step kernel (nvcc otherwise outlines the large
// ones with a stack frame)
#define AI __attribute__((always_inline))
#ifndef MRLBM_Q27_PRODUCT
#define MRLBM_Q27_PRODUCT 1
#endif
constexpr bool Q27_PRODUCT = MRLBM_Q27_PRODUCT;
#ifndef MRLBM_ROTATE_PAIRED
#define MRLBM_ROTATE_PAIRED 0
#endif
constexpr bool ROTATE = MRLBM_ROTATE_PAIRED;

// ------------------------------------------------------------ pairs over c_m = (-1, +1)
template <typename Real> struct Pr;
template <> struct __align__(8) Pr<float> {
    float2 v;
    __device__ __forceinline__ float lo() const { return v.x; }
    __device__ __forceinline__ float hi() const { return v.y; }
};
// fp64: two independent registers (no 128-bit alignment: DFMA has no packed
// form, and aligned quads would cost register moves), two 64-bit smem accesses
struct D2 {
    double x, y;
};
template <> struct Pr<double> {
    D2 v;
    __device__ __forceinline__ double lo() const { return v.x; }
    __device__ __forceinline__ double hi() const { return v.y; }
};
__device__ __forceinline__ Pr<float> mkpr(float l, float h) { return {make_float2(l, h)}; }
__device__ __forceinline__ Pr<double> mkpr(double l, double h) { return {D2{l, h}}; }
__device__ __forceinline__ Pr<float> operator+(Pr<float> a, Pr<float> b) { return {__fadd2_rn(a.v, b.v)}; }
__device__ __forceinline__ Pr<double> operator+(Pr<double> a, Pr<double> b) { return mkpr(a.v.x + b.v.x, a.v.y + b.v.y); }
__device__ __forceinline__ Pr<float> operator-(Pr<float> a, Pr<float> b)
{
    return {__ffma2_rn(b.v, make_float2(-1.0f, -1.0f), a.v)};
}
__device__ __forceinline__ Pr<double> operator-(Pr<double> a, Pr<double> b) { return mkpr(a.v.x - b.v.x, a.v.y - b.v.y); }
__device__ __forceinline__ Pr<float> operator-(Pr<float> a) { return {__fmul2_rn(a.v, make_float2(-1.0f, -1.0f))}; }
__device__ __forceinline__ Pr<double> operator-(Pr<double> a) { return mkpr(-a.v.x, -a.v.y); }

// generic value ops for V = Real or Pr<Real>; c is a (compile-time) scalar
__device__ __forceinline__ float vfma(float c, float x, float y) { return fmaf(c, x, y); }
__device__ __forceinline__ double vfma(double c, double x, double y) { return fma(c, x, y); }
__device__ __forceinline__ Pr<float> vfma(float c, Pr<float> x, Pr<float> y) { return {__ffma2_rn(make_float2(c, c), x.v, y.v)}; }
__device__ __forceinline__ Pr<double> vfma(double c, Pr<double> x, Pr<double> y)
{
    return mkpr(fma(c, x.v.x, y.v.x), fma(c, x.v.y, y.v.y));
}
__device__ __forceinline__ float vmul(float c, float x) { return c * x; }
__device__ __forceinline__ double vmul(double c, double x) { return c * x; }
__device__ __forceinline__ Pr<float> vmul(float c, Pr<float> x) { return {__fmul2_rn(make_float2(c, c), x.v)}; }
__device__ __forceinline__ Pr<double> vmul(double c, Pr<double> x) { return mkpr(c * x.v.x, c * x.v.y); }
template <typename Real> __device__ __forceinline__ Real vzero(Real *) { return Real(0); }
template <typename Real> __device__ __forceinline__ Pr<Real> vzero(Pr<Real> *) { return mkpr(Real(0), Real(0)); }
// s * x + y with the scalar s broadcast (x, y pairs)
__device__ __forceinline__ Pr<float> pfma_b(float s, Pr<float> x, Pr<float> y) { return {__ffma2_rn(make_float2(s, s), x.v, y.v)}; }
__device__ __forceinline__ Pr<double> pfma_b(double s, Pr<double> x, Pr<double> y)
{
    return mkpr(fma(s, x.v.x, y.v.x), fma(s, x.v.y, y.v.y));
}
// c * x + q with the constant c and the scalar q broadcast
__device__ __forceinline__ Pr<float> pfma_cb(float c, Pr<float> x, float q) { return {__ffma2_rn(make_float2(c, c), x.v, make_float2(q, q))}; }
__device__ __forceinline__ Pr<double> pfma_cb(double c, Pr<double> x, double q) { return mkpr(fma(c, x.v.x, q), fma(c, x.v.y, q)); }
// (S - h x1, S + h x1): one packed FMA with both scalars broadcast
__device__ __forceinline__ Pr<float> pm_pair(float h, float x1, float S)
{
    return {__ffma2_rn(make_float2(x1, x1), make_float2(-h, h), make_float2(S, S))};
}
__device__ __forceinline__ Pr<double> pm_pair(double h, double x1, double S) { return mkpr(fma(-h, x1, S), fma(h, x1, S)); }

// ------------------------------------------------------------ synthesis on scalars or pairs
// One 1D synthesis maps the coefficients (x0, x1, x2) of orders 0, 1, 2 along
// an axis to the values at c = -1, 0, +1:
//   g0 = c0 x0 + k02 x2,   S = x0 + c2 x2,   g+- = S +- h x1
// SYN_W   weighted, coefficients carry tscale (RECON_TENSOR_W, as synth_p)
// SYN_U36 unweighted, coefficients carry only 1/36: the per-axis Hermite scale
//         s = (1, 3, 3/2) (hscale = prod_a s(h_a)) and He'_2(0) = -1,
//         He'_2(+-1) = 2 give c0 = 1, k02 = -3/2, c2 = 3, h = 3 (D3Q19, with
//         collide_u36; f_i = (36 w_i) V afterwards)
enum { SYN_W = 0, SYN_U36 = 1 };
template <int MODE, typename Real> struct SynC {
    static constexpr Real c0 = MODE == SYN_W ? Real(4) : Real(1);
    static constexpr Real k02 = MODE == SYN_W ? Real(-1) : Real(-1.5);
    static constexpr Real c2 = MODE == SYN_W ? Real(0.5) : Real(3);
    static constexpr Real h = MODE == SYN_W ? Real(0.5) : Real(3);
};
// One 1D synthesis with compile-time absent inputs, on V (Real or Pr<Real>).
template <int MODE, bool P0, bool P1, bool P2, typename Real, typename V>
__device__ __forceinline__ void synth_v(V x0, V x1, V x2, V &gm, V &g0, V &gp)
{
    using K = SynC<MODE, Real>;
    V S;
    if constexpr (P0 && P2) {
        S = vfma(K::c2, x2, x0);
        if constexpr (K::c0 == Real(1)) g0 = vfma(K::k02, x2, x0);
        else g0 = vfma(K::c0, x0, -x2);
    } else if constexpr (P0) {
        S = x0;
        if constexpr (K::c0 == Real(1)) g0 = x0;
        else g0 = vmul(K::c0, x0);
    } else if constexpr (P2) {
        S = vmul(K::c2, x2);
        if constexpr (K::k02 == Real(-1)) g0 = -x2;
        else g0 = vmul(K::k02, x2);
    }
    if constexpr (P1 && (P0 || P2)) { gp = vfma(K::h, x1, S); gm = vfma(-K::h, x1, S); }
    else if constexpr (P1) { gp = vmul(K::h, x1); gm = vmul(-K::h, x1); }
    else if constexpr (P0 || P2) { gp = S; gm = S; }
    else { gp = gm = vzero((V *)nullptr); }
    if constexpr (!(P0 || P2)) g0 = vzero((V *)nullptr);
}

// The z step on scalar coefficients: g0 (c_z = 0) and the pair (c_z = -1, +1).
template <int MODE, bool P0, bool P1, bool P2, typename Real>
__device__ __forceinline__ void zsynth(Real x0, Real x1, Real x2, Real &g0, Pr<Real> &gpm)
{
    using K = SynC<MODE, Real>;
    Real S = Real(0);
    if constexpr (P0 && P2) {
        S = fma(K::c2, x2, x0);
        if constexpr (K::c0 == Real(1)) g0 = fma(K::k02, x2, x0);
        else g0 = fma(K::c0, x0, -x2);
    } else if constexpr (P0) {
        S = x0;
        g0 = K::c0 == Real(1) ? x0 : K::c0 * x0;
    } else if constexpr (P2) {
        S = K::c2 * x2;
        g0 = K::k02 * x2;
    } else {
        g0 = Real(0);
    }
    if constexpr (P1) gpm = pm_pair(K::h, x1, S);
    else gpm = mkpr(S, S);
}

// Eq 14 (3D, sum-factorised; RECON_TENSOR_W / RECON_TENSOR_U as in
// reconstruct_tensor3): shifted post-collision populations as
//   f0[ca+1][cb+1]  = f~*(ca, cb, 0)                  (scalars)
//   fp[ca+1][cb+1]  = (f~*(ca, cb, -1), f~*(ca, cb, +1))  (pairs)
// Entries of directions the lattice lacks are never read (dead code).
template <int LAT, bool REC, typename Real>
__device__ __forceinline__ void reconstruct_pairs(const Real (&A)[Basis<LAT, REC>::NH], Real (&f0)[3][3], Pr<Real> (&fp)[3][3])
{
    using L = Lattice<LAT>;
    constexpr bool W = recon_kind<LAT, REC>() == RECON_TENSOR_W;
    constexpr int MODE = W ? SYN_W : SYN_U36;
    auto coef = [&](auto kc) -> Real {
        constexpr int k = decltype(kc)::value;
        if constexpr (k < 0) return Real(0);
        else return A[k];
    };
    Real T0[3][3];     // [h_x][h_y], c_z = 0
    Pr<Real> Tp[3][3]; // [h_x][h_y], c_z = -1 / +1
    static_for<0, 9>([&](auto abk) {
        constexpr int a = decltype(abk)::value / 3, b = decltype(abk)::value % 3;
        constexpr int k0 = hindex<LAT, REC>(a, b, 0), k1 = hindex<LAT, REC>(a, b, 1), k2 = hindex<LAT, REC>(a, b, 2);
        zsynth<MODE, (k0 >= 0), (k1 >= 0), (k2 >= 0), Real>(coef(std::integral_constant<int, k0>{}),
                                                        coef(std::integral_constant<int, k1>{}),
                                                        coef(std::integral_constant<int, k2>{}), T0[a][b], Tp[a][b]);
    });
    Real U0[3][3];     // [h_x][c_y + 1]
    Pr<Real> Up[3][3];
    static_for<0, 3>([&](auto ak) {
        constexpr int a = decltype(ak)::value;
        synth_v<MODE, presT<LAT, REC>(a, 0, 0), presT<LAT, REC>(a, 1, 0), presT<LAT, REC>(a, 2, 0), Real>(
            T0[a][0], T0[a][1], T0[a][2], U0[a][0], U0[a][1], U0[a][2]);
        synth_v<MODE, presT<LAT, REC>(a, 0, 1), presT<LAT, REC>(a, 1, 1), presT<LAT, REC>(a, 2, 1), Real>(
            Tp[a][0], Tp[a][1], Tp[a][2], Up[a][0], Up[a][1], Up[a][2]);
    });
    static_for<0, 3>([&](auto yk) {
        constexpr int yi = decltype(yk)::value;
        Real V0[3];
        Pr<Real> Vp[3];
        synth_v<MODE, presU<LAT, REC>(0, yi - 1, 0), presU<LAT, REC>(1, yi - 1, 0), presU<LAT, REC>(2, yi - 1, 0), Real>(
            U0[0][yi], U0[1][yi], U0[2][yi], V0[0], V0[1], V0[2]);
        synth_v<MODE, presU<LAT, REC>(0, yi - 1, 1), presU<LAT, REC>(1, yi - 1, 1), presU<LAT, REC>(2, yi - 1, 1), Real>(
            Up[0][yi], Up[1][yi], Up[2][yi], Vp[0], Vp[1], Vp[2]);
        static_for<0, 3>([&](auto xk) {
            constexpr int xi = decltype(xk)::value;
            if constexpr (W) {
                f0[xi][yi] = V0[xi];
                fp[xi][yi] = Vp[xi];
            } else {
                // D3Q19 weights are not products: f = (36 w) V, 36 w in {12, 2, 1}
                constexpr int k0 = dir_of<L>(xi - 1, yi - 1, 0), k1 = dir_of<L>(xi - 1, yi - 1, 1);
                constexpr int m0 = k0 >= 0 ? int(L::w[k0] * 36.0 + 0.5) : 1;
                constexpr int m1 = k1 >= 0 ? int(L::w[k1] * 36.0 + 0.5) : 1;
                if constexpr (m0 == 1) f0[xi][yi] = V0[xi];
                else if constexpr (m0 == 2) f0[xi][yi] = V0[xi] + V0[xi];
                else f0[xi][yi] = Real(m0) * V0[xi];
                if constexpr (m1 == 1) fp[xi][yi] = Vp[xi];
                else if constexpr (m1 == 2) fp[xi][yi] = Vp[xi] + Vp[xi];
                else fp[xi][yi] = vmul(Real(m1), Vp[xi]);
            }
        });
    });
}

// ------------------------------------------------------------ D3Q27 recursive in product form
// For the full tensor basis the recursive-regularized coefficients are (eqs
// 10, 12-13; R8)  a*_h = rho u^h + (omega/2) sum_ab Pneq_ab d_a d_b u^h  for
// every h in {0,1,2}^3 (the pair-sum closed form is this second derivative),
// and the weighted Hermite synthesis (eq 14) is a tensor product of 1D maps.
// So every term is separable and the synthesis of each factor is a 1D
// function of one velocity component:
//   E(c) = syn(1, u, u^2):  E(0) = 2/3 - u^2,  E(+-1) = 1/6 + u^2/2 +- u/2
//   D(c) = syn(0, 1, 2u):   D(0) = -2u,        D(+-1) = u +- 1/2
//   DD(c)= syn(0, 0, 2):    DD(0) = -2,        DD(+-1) = 1
// (D1Q3 weights w(0) = 2/3, w(1) = 1/6 and the Hermite scales folded in), and
//   f* = rho ExEyEz + (omega/2)(Pxx DDx Ey Ez + Pyy Ex DDy Ez + Pzz Ex Ey DDz)
//        + omega (Pxy Dx Dy Ez + Pxz Dx Ey Dz + Pyz Ex Dy Dz).
// The state is shifted (R16): f~ = f* - Wx Wy Wz with W = E(u = 0); writing
// E = W + Ehat and rho = 1 + drho, rho ExEyEz - WxWyWz
//   = [(drho Ex + Ehatx) Ey + Wx Ehaty] Ez + Wx Wy Ehatz   (small terms only).
// Evaluated x first, then per (cx, cy), then the c_z pair / scalar -- it
// replaces collide_coeffs + reconstruct_pairs for D3Q27 recursive in fp64
// (209 instead of 262 FP64 instructions per node) and gives the same
// populations up to rounding.  Not in fp32: E(+-1) = 1/6 + u^2/2 +- u/2 stored
// as one fp32 number keeps only ~1.5e-8 of its O(u) part, and the 1000-step
// parity error grows 3-6x (profiles/r03/probe.txt); keeping the weight and the
// small part apart costs as many instructions as the sum-factorised form.
template <typename Real>
__device__ __forceinline__ void collide_reconstruct_q27r(const Real (&m)[10], Real omega, Real (&f0)[3][3], Pr<Real> (&fp)[3][3])
{
    const Real drho = m[0];
    const Real rho = Real(1) + drho;
    const Real u[3] = {m[1], m[2], m[3]};
    // Pi^neq = Pi - rho u u; halves of the diagonal times omega, off-diagonal times omega
    const Real ru0 = rho * u[0], ru1 = rho * u[1], ru2 = rho * u[2];
    const Real hw = Real(0.5) * omega;
    const Real hPxx = hw * fma(-ru0, u[0], m[4]), hPyy = hw * fma(-ru1, u[1], m[5]), hPzz = hw * fma(-ru2, u[2], m[6]);
    const Real wPxy = omega * fma(-ru0, u[1], m[7]), wPxz = omega * fma(-ru0, u[2], m[8]), wPyz = omega * fma(-ru1, u[2], m[9]);
    // per-axis 1D factors, index c + 1
    Real E[3][3], Eh[3][3], Dv[3][3];
#pragma unroll
    for (int a = 0; a < 3; a++) {
        const Real uu = u[a] * u[a];
        const Real h2 = Real(0.5) * uu;
        Eh[a][1] = -uu;
        Eh[a][0] = fma(Real(-0.5), u[a], h2);
        Eh[a][2] = fma(Real(0.5), u[a], h2);
        E[a][1] = Real(2.0 / 3.0) - uu;
        E[a][0] = Real(1.0 / 6.0) + Eh[a][0];
        E[a][2] = Real(1.0 / 6.0) + Eh[a][2];
        Dv[a][1] = Real(-2) * u[a];
        Dv[a][0] = u[a] - Real(0.5);
        Dv[a][2] = u[a] + Real(0.5);
    }
    const Pr<Real> Ez = mkpr(E[2][0], E[2][2]), Dz = mkpr(Dv[2][0], Dv[2][2]), Ehz = mkpr(Eh[2][0], Eh[2][2]);
    static_for<0, 3>([&](auto xk) {
        constexpr int xi = decltype(xk)::value;
        constexpr Real Wx = xi == 1 ? Real(2.0 / 3.0) : Real(1.0 / 6.0);
        constexpr Real DDx = xi == 1 ? Real(-2) : Real(1);
        const Real ax = fma(drho, E[0][xi], Eh[0][xi]);  // rho Ex - Wx
        const Real al = fma(DDx, hPxx, ax);               // + (omega/2) Pxx DDx
        const Real be = hPyy * E[0][xi];
        const Real ga = wPxy * Dv[0][xi];
        const Real ze = hPzz * E[0][xi];
        const Real de = wPxz * Dv[0][xi];
        const Real ep = wPyz * E[0][xi];
        static_for<0, 3>([&](auto yk) {
            constexpr int yi = decltype(yk)::value;
            constexpr Real Wy = yi == 1 ? Real(2.0 / 3.0) : Real(1.0 / 6.0);
            constexpr Real DDy = yi == 1 ? Real(-2) : Real(1);
            constexpr Real WW = Wx * Wy;
            const Real Q1 = fma(E[1][yi], al, fma(Wx, Eh[1][yi], fma(DDy, be, ga * Dv[1][yi])));
            const Real Q2 = ze * E[1][yi];
            const Real Q3 = fma(de, E[1][yi], ep * Dv[1][yi]);
            // c_z = 0: Q1 Ez0 - 2 Q2 + Q3 Dz0 + Wx Wy Ehatz0
            f0[xi][yi] = fma(Q1, E[2][1], fma(Real(-2), Q2, fma(Q3, Dv[2][1], WW * Eh[2][1])));
            // c_z = -1, +1: Q1 Ez + Q2 + Q3 Dz + Wx Wy Ehatz
            fp[xi][yi] = pfma_b(Q1, Ez, pfma_b(Q3, Dz, pfma_cb(WW, Ehz, Q2)));
        });
    });
}

// ------------------------------------------------------------ D3Q27 recursive, regrouped
// The 27 post-collision coefficients of D3Q27 recursive for the weighted
// synthesis (SYN_W: A_h = tscale(h) a*_h, tscale = 6^-(#axes with h = 0)),
// with the pair sums of the recursion (eqs 12-13, R8) regrouped so that each
// order reuses the one below (as collide_u36 for D3Q19).  With
// S_ab = Pi*_ab = rho u_a u_b + omega P_ab (P = Pi^neq), R_ab = 2 omega P_ab:
//   a210 = uy S_xx + ux R_xy                      a111 = uz S_xy + (uy R_xz + ux R_yz)/2
//   a220 = uy a210 + ux (omega P_yy ux + R_xy uy) a211 = uz a210 + ux (R_xz uy + omega P_yz ux)
//   a221 = uz a220 + ux uy (uy R_xz + ux R_yz)    a222 = uz a221 + ux uy (omega P_zz ux uy + uz (uy R_xz + ux R_yz))
// and their permutations (each identity is the pair-sum closed form of
// collide_coeffs, term by term).  ~105 instead of 154 FP32 instructions.
template <typename Real>
__device__ __forceinline__ void collide_q27r(const Real (&m)[10], Real omega, Real (&A)[27])
{
    constexpr Real t1 = Real(1.0 / 6.0), t2 = Real(1.0 / 36.0), t3 = Real(1.0 / 216.0);
    const Real drho = m[0];
    const Real rho = Real(1) + drho;
    const Real ux = m[1], uy = m[2], uz = m[3];
    const Real rx = rho * ux, ry = rho * uy, rz = rho * uz;
    const Real rxx = rx * ux, ryy = ry * uy, rzz = rz * uz, rxy = rx * uy, rxz = rx * uz, ryz = ry * uz;
    const Real Pxx = m[4] - rxx, Pyy = m[5] - ryy, Pzz = m[6] - rzz;
    const Real Pxy = m[7] - rxy, Pxz = m[8] - rxz, Pyz = m[9] - ryz;
    const Real wxx = omega * Pxx, wyy = omega * Pyy, wzz = omega * Pzz;
    const Real w2 = omega + omega;
    const Real Rxy = w2 * Pxy, Rxz = w2 * Pxz, Ryz = w2 * Pyz;
    const Real wxy = omega * Pxy, wxz = omega * Pxz, wyz = omega * Pyz;
    const Real Sxx = rxx + wxx, Syy = ryy + wyy, Szz = rzz + wzz;
    const Real Sxy = rxy + wxy, Sxz = rxz + wxz, Syz = ryz + wyz;
    const Real a210 = fma(uy, Sxx, ux * Rxy), a201 = fma(uz, Sxx, ux * Rxz);
    const Real a120 = fma(ux, Syy, uy * Rxy), a021 = fma(uz, Syy, uy * Ryz);
    const Real a102 = fma(ux, Szz, uz * Rxz), a012 = fma(uy, Szz, uz * Ryz);
    const Real tyz = fma(uy, Rxz, ux * Ryz); // uy R_xz + ux R_yz
    const Real a111 = fma(uz, Sxy, Real(0.5) * tyz);
    const Real a220 = fma(ux, fma(wyy, ux, Rxy * uy), uy * a210);
    const Real a202 = fma(ux, fma(wzz, ux, Rxz * uz), uz * a201);
    const Real a022 = fma(uy, fma(wzz, uy, Ryz * uz), uz * a021);
    const Real a211 = fma(uz, a210, ux * fma(Rxz, uy, wyz * ux));
    const Real a121 = fma(uz, a120, uy * fma(Ryz, ux, wxz * uy));
    const Real a112 = fma(uy, a102, uz * fma(Ryz, ux, wxy * uz));
    const Real uxy = ux * uy, uxz = ux * uz, uyz = uy * uz;
    const Real a221 = fma(uz, a220, uxy * tyz);
    const Real a212 = fma(uy, a202, uxz * fma(uz, Rxy, ux * Ryz));
    const Real a122 = fma(ux, a022, uyz * fma(uz, Rxy, uy * Rxz));
    const Real a222 = fma(uz, a221, uxy * fma(wzz, uxy, uz * tyz));
    // basis order (lattice.cuh), times tscale
    A[0] = t3 * drho;
    A[1] = t2 * rx;
    A[2] = t2 * ry;
    A[3] = t2 * rz;
    A[4] = t2 * Sxx;
    A[5] = t2 * Syy;
    A[6] = t2 * Szz;
    A[7] = t1 * Sxy;
    A[8] = t1 * Sxz;
    A[9] = t1 * Syz;
    A[10] = t1 * a210;
    A[11] = t1 * a201;
    A[12] = t1 * a120;
    A[13] = t1 * a021;
    A[14] = t1 * a102;
    A[15] = t1 * a012;
    A[16] = a111;
    A[17] = t1 * a220;
    A[18] = t1 * a202;
    A[19] = t1 * a022;
    A[20] = a211;
    A[21] = a121;
    A[22] = a112;
    A[23] = a221;
    A[24] = a212;
    A[25] = a122;
    A[26] = a222;
}

// ------------------------------------------------------------ exchange-plane slots
// In-plane movers along B (c_b != 0) go through shared memory: the pairs
// (c_m = +-1) and the c_m = 0 scalars each get one slot per (c_a, c_b).
template <class L> struct Slots3 {
    static constexpr bool haspair(int ca, int cb) { return dir_of<L>(ca, cb, 1) >= 0; }
    static constexpr bool hasz(int ca, int cb) { return dir_of<L>(ca, cb, 0) >= 0; }
    static constexpr int pslot(int ca, int cb)
    {
        int s = 0;
        for (int b = -1; b <= 1; b += 2)
            for (int a = -1; a <= 1; a++) {
                if (a == ca && b == cb) return haspair(a, b) ? s : -1;
                s += haspair(a, b) ? 1 : 0;
            }
        return -1;
    }
    static constexpr int zslot(int ca, int cb)
    {
        int s = 0;
        for (int b = -1; b <= 1; b += 2)
            for (int a = -1; a <= 1; a++) {
                if (a == ca && b == cb) return hasz(a, b) ? s : -1;
                s += hasz(a, b) ? 1 : 0;
            }
        return -1;
    }
    static constexpr int count(bool pair)
    {
        int s = 0;
        for (int b = -1; b <= 1; b += 2)
            for (int a = -1; a <= 1; a++) s += (pair ? haspair(a, b) : hasz(a, b)) ? 1 : 0;
        return s;
    }
    static constexpr int NP = count(true), NZ = count(false);
};

template <int LAT, typename Real, int TB, int S> struct Step3Smem {
    using L = Lattice<LAT>;
    using SL = Slots3<L>;
    static constexpr int TA = 32, NT = TA * TB;
    static constexpr int AL = 16 / int(sizeof(Real));
    static constexpr int BW = (TA + AL - 1 + AL - 1) / AL * AL;
    static constexpr size_t box_elems = size_t(L::M) * TB * BW;
    static constexpr size_t stage_elems = (box_elems * sizeof(Real) + 127) / 128 * 128 / sizeof(Real);
    // one exchange plane: NP pair slots then NZ scalar slots (NT entries each)
    static constexpr size_t plane_bytes = (size_t(SL::NP) * NT * 2 + size_t(SL::NZ) * NT) * sizeof(Real);
    static constexpr size_t bytes = S * stage_elems * sizeof(Real) + 2 * plane_bytes + (S + 4) * sizeof(uint64_t) + 128;
};

// ------------------------------------------------------------ column sums of one pulled group
template <class A, class B, class C, class D, class E, class F> struct Cols {
    A S;   // sum f
    B Sa;  // sum c_a f
    C Sb;  // sum c_b f
    D Saa; // sum c_a^2 f
    E Sbb; // sum c_b^2 f
    F Sab; // sum c_a c_b f
};
template <class A, class B, class C, class D, class E, class F>
__device__ __forceinline__ Cols<A, B, C, D, E, F> mkcols(A S, B Sa, C Sb, D Saa, E Sbb, F Sab)
{
    return {S, Sa, Sb, Saa, Sbb, Sab};
}
// G(ia, ib) -> OV<present, V>: the arrivals of one c_m group; sums over c_a per
// row c_b, then over c_b (sum-factorised, as accum_group)
template <class GF> __device__ __forceinline__ auto colsums(GF &&G)
{
    using I0 = std::integral_constant<int, 0>;
    using I1 = std::integral_constant<int, 1>;
    using I2 = std::integral_constant<int, 2>;
    auto rm = sums3(G(I0{}, I0{}), G(I1{}, I0{}), G(I2{}, I0{}));
    auto rz = sums3(G(I0{}, I1{}), G(I1{}, I1{}), G(I2{}, I1{}));
    auto rp = sums3(G(I0{}, I2{}), G(I1{}, I2{}), G(I2{}, I2{}));
    auto Sbb = ov_add(rp.r0, rm.r0);
    auto Sb = ov_sub(rp.r0, rm.r0);
    auto S = ov_add(Sbb, rz.r0);
    auto Sa = ov_add(ov_add(rp.r1, rm.r1), rz.r1);
    auto Saa = ov_add(ov_add(rp.r2, rm.r2), rz.r2);
    auto Sab = ov_sub(rp.r1, rm.r1);
    return mkcols(S, Sa, Sb, Saa, Sbb, Sab);
}
template <bool HI, bool P, typename Real> __device__ __forceinline__ OV<P, Real> half(OV<P, Pr<Real>> x)
{
    if constexpr (P) return OV<true, Real>{HI ? x.v.hi() : x.v.lo()};
    else return OV<false, Real>{};
}
// acc += (or =, AS) the raw moments of a group moving by CM along C (3D slots)
template <int CM, bool AS, typename Real, class C> __device__ __forceinline__ void acc_cols(Real (&acc)[10], const C &c)
{
    constexpr int CM2 = CM * CM;
    ov_acc<1, AS>(acc[0], c.S);
    ov_acc<1, AS>(acc[1], c.Sa);
    ov_acc<1, AS>(acc[2], c.Sb);
    ov_acc<CM, AS>(acc[3], c.S);
    ov_acc<1, AS>(acc[pslot<3>(0, 0)], c.Saa);
    ov_acc<1, AS>(acc[pslot<3>(1, 1)], c.Sbb);
    ov_acc<CM2, AS>(acc[pslot<3>(2, 2)], c.S);
    ov_acc<1, AS>(acc[pslot<3>(0, 1)], c.Sab);
    ov_acc<CM, AS>(acc[pslot<3>(0, 2)], c.Sa);
    ov_acc<CM, AS>(acc[pslot<3>(1, 2)], c.Sb);
}
template <bool HI, class C> __device__ __forceinline__ auto cols_half(const C &c)
{
    return mkcols(half<HI>(c.S), half<HI>(c.Sa), half<HI>(c.Sb), half<HI>(c.Saa), half<HI>(c.Sbb), half<HI>(c.Sab));
}

// ------------------------------------------------------------ step kernel (3D, paired)
// SPLIT: split-phase exchange barriers instead of one __syncthreads per layer.
// Each warp arrives on xfull[plane] after publishing its movers and waits on
// it only before pulling (rows that do not pull -- the halo rows -- never
// wait); it arrives on xempty[plane] after its last read of the plane, and a
// warp waits on xempty only before it overwrites the plane two layers later.
// Warps may then run up to a layer apart, so the collide/reconstruct phase of
// some overlaps the pull phase of others (one CTA per SM otherwise phase-locks
// all its warps onto one pipe at a time).
__device__ __forceinline__ void mbar_arrive(uint64_t *bar)
{
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

template <int LAT, bool REC, typename Real, int TB, int S, int MINB, bool PUSH = false, bool SPLIT = false, bool ONEBODY = false>
__global__ void __launch_bounds__(32 * TB, MINB) mrlbm_step3_kernel(const __grid_constant__ CUtensorMap tmap,
                                                                   const StepArgs p)
{
    using L = Lattice<LAT>;
    using X = Axes<L>;
    using SL = Slots3<L>;
    using SM = Step3Smem<LAT, Real, TB, S>;
    static_assert(L::D == 3, "3D kernel");
    constexpr int M = L::M, TA = 32, NT = TA * TB;
    constexpr int NP = SL::NP;

    extern __shared__ __align__(128) unsigned char smem_raw[];
    Real *stage = reinterpret_cast<Real *>(smem_raw);
    unsigned char *planes = reinterpret_cast<unsigned char *>(stage + S * SM::stage_elems);
    uint64_t *full = reinterpret_cast<uint64_t *>(planes + 2 * SM::plane_bytes);
    uint64_t *xfull = full + S, *xempty = full + S + 2; // SPLIT only

    const int tid = threadIdx.x;
    const int tx = tid % TA, ty = tid / TA;
    // launch order: groups of rastG B-tiles (see mrlbm_step_kernel)
    int tA = blockIdx.x, tBi = blockIdx.y;
    if (p.rastG > 0) {
        const int Lx = blockIdx.x;
        const int span = p.rastG * p.tilesA;
        const int grp = Lx / span;
        const int w = Lx - grp * span;
        const int g0 = grp * p.rastG;
        const int gsz = min(p.rastG, p.tilesB - g0);
        tA = w / gsz;
        tBi = g0 + (w - tA * gsz);
    }
    const int a0 = tA * (TA - 2) - 1;
    const int b0 = tBi * (TB - 2) - 1;
    const int a = a0 + tx, b = b0 + ty;
    const int nA = p.nA, nB = p.nB, nC = p.nC;

    const bool second = (int)blockIdx.z >= p.nseg1;
    const int c0 = second ? p.c2_begin + ((int)blockIdx.z - p.nseg1) * p.seg_len : p.c_begin + blockIdx.z * p.seg_len;
    const int c1 = min(c0 + p.seg_len, second ? p.c2_end : p.c_end);
    if (c0 >= c1) return;
    const int boxA = ((a0 + p.padA) / SM::AL) * SM::AL;
    const int offA = a0 + p.padA - boxA;
    const int cfirst = (c0 > 0 || p.lo_nb) ? c0 - 1 : c0;
    const int clast = (c1 < nC || p.hi_nb) ? c1 : c1 - 1;
    const int nl = clast - cfirst + 1;

    // ---- per-thread roles (see mrlbm_step_kernel; every window position is
    // computed: positions without a node hold zero moments -> zero populations)
    const bool perA = p.kind[0] == BC_PERIODIC, perB = p.kind[2] == BC_PERIODIC;
    const bool inA = a >= 0 && a < nA, inB = b >= 0 && b < nB;
    const bool rowlane = ty >= 1 && ty <= TB - 2; // rows that pull (all 32 lanes: shuffles)
    const bool owner = rowlane && tx >= 1 && tx < TA - 1 && inA && inB;
    const bool cta_open = (p.kind[0] >= BC_VELOCITY && a0 < 0) || (p.kind[1] >= BC_VELOCITY && a0 + TA - 1 >= nA - 1) ||
                          (p.kind[2] >= BC_VELOCITY && b0 <= 0) || (p.kind[3] >= BC_VELOCITY && b0 + TB - 1 >= nB - 1);
    const int gA = !perA ? 0 : (a == 0 ? nA : (a == nA - 1 ? -nA : 0));
    const int gB = !perB ? 0 : (b == 0 ? nB : (b == nB - 1 ? -nB : 0));
    auto is_wall = [](int k) AI { return k == BC_WALL || k == BC_MOVING; };
    const int bbA = (a == 0 && is_wall(p.kind[0])) ? -1 : ((a == nA - 1 && is_wall(p.kind[1])) ? 1 : 0);
    const int bbB = (b == 0 && is_wall(p.kind[2])) ? -1 : ((b == nB - 1 && is_wall(p.kind[3])) ? 1 : 0);
    int openF = -1, nx_in = 0, ny_in = 0;
    if (owner) {
        if (a == 0 && p.kind[0] >= BC_VELOCITY) { openF = 0; nx_in = 1; }
        else if (a == nA - 1 && p.kind[1] >= BC_VELOCITY) { openF = 1; nx_in = -1; }
        else if (b == 0 && p.kind[2] >= BC_VELOCITY) { openF = 2; ny_in = 1; }
        else if (b == nB - 1 && p.kind[3] >= BC_VELOCITY) { openF = 3; ny_in = -1; }
    }
    // C walls at this rank's global ends (the layer test is per layer)
    const bool wallClo = !p.lo_nb, wallChi = !p.hi_nb;

    Real *dst = reinterpret_cast<Real *>(p.dst);
    const Real omega = Real(p.omega);
    auto plane_of = [&](int c) AI -> int { return p.wrapC ? ((c % nC + nC) % nC) + 1 : c + 1; };

    // ---- TMA ring prologue
    if (tid == 0) {
        prefetch_tmap(&tmap);
#pragma unroll
        for (int s = 0; s < S; s++) mbar_init(&full[s], 1);
        if constexpr (SPLIT) {
            for (int q = 0; q < 2; q++) {
                mbar_init(&xfull[q], TB);
                mbar_init(&xempty[q], TB);
            }
        }
        fence_barrier_init();
    }
    __syncthreads();
    constexpr uint32_t stage_bytes = uint32_t(SM::box_elems * sizeof(Real));
    if (tid == 0) {
        for (int s = 0; s < S && s < nl; s++) {
            mbar_expect_tx(&full[s], stage_bytes);
            tma_load_4d(stage + s * SM::stage_elems, &tmap, &full[s], boxA, b0 + p.padB, 0, plane_of(cfirst + s));
        }
    }

    Real accA[M], accB[M], accC[M];
#pragma unroll
    for (int q = 0; q < M; q++) {
        accA[q] = Real(0);
        accB[q] = Real(0);
        accC[q] = Real(0);
    }

    Real *const dst_node = dst + (long long)b * p.pitch + a;
    auto finalize_store = [&](const Real (&s)[M], int c) AI {
        Real out[M];
        const Real S0 = s[0];
        if (openF < 0) {
            const Real inv = rcp_nr(Real(1) + S0);
            out[0] = S0;
#pragma unroll
            for (int q = 0; q < 3; q++) out[1 + q] = s[1 + q] * inv;
#pragma unroll
            for (int q = 0; q < 3; q++)
#pragma unroll
                for (int r = q; r < 3; r++)
                    out[pslot<3>(q, r)] = (q == r) ? fma(S0, Real(-1.0 / 3.0), s[pslot<3>(q, r)]) : s[pslot<3>(q, r)];
        } else {
            RVec<Real, M> sv;
#pragma unroll
            for (int q = 0; q < M; q++) sv.v[q] = s[q];
            const RVec<Real, M> ov = finalize_open<LAT, Real>(sv, openF, nx_in, ny_in, c + p.c_offset, a, b, nA, nB, &p);
#pragma unroll
            for (int q = 0; q < M; q++) out[q] = ov.v[q];
        }
        if (!owner) return;
        auto store_plane = [&](Real *o) AI {
            const int ms = int(p.mstride); // < 2^31 elements per moment plane
#pragma unroll
            for (int q = 0; q < M; q++) o[q * ms] = out[q];
            if (gA | gB) {
                auto put = [&](int da, int db) AI {
                    Real *g = o + (long long)db * p.pitch + da;
#pragma unroll
                    for (int q = 0; q < M; q++) g[q * ms] = out[q];
                };
                if (gA) put(gA, 0);
                if (gB) put(0, gB);
                if (gA && gB) put(gA, gB);
            }
        };
        store_plane(dst_node + (long long)(c + 1) * p.pstride);
        if constexpr (PUSH) {
            void *peer = (c == 0) ? p.peer_lo : ((c == nC - 1) ? p.peer_hi : nullptr);
            if (peer) {
                store_plane(reinterpret_cast<Real *>(peer) + (long long)b * p.pitch + a);
                __threadfence_system();
            }
        }
    };

    // one layer: on entry X holds layer c-1 and Y layer c; on exit Y holds
    // layer c and Z layer c+1 (Z = X in the two-set scheme)
    // produce(it): collide + reconstruct layer it and publish its c_b != 0 movers
    // into plane it & 1; the own c_b = 0 row stays in registers (f0, fp)
    auto produce = [&](const int it, Real (&f0)[3][3], Pr<Real> (&fp)[3][3], Real &rho_own) AI {
        const int s = it % S;
        mbar_wait(&full[s], (it / S) & 1);
        Real m[M];
        {
            const Real *st = stage + s * SM::stage_elems + ty * SM::BW + tx + offA;
#pragma unroll
            for (int q = 0; q < M; q++) m[q] = st[q * (TB * SM::BW)];
        }
        unsigned char *Fl = planes + (it & 1) * SM::plane_bytes;
        Pr<Real> *Fp = reinterpret_cast<Pr<Real> *>(Fl);
        Real *Fz = reinterpret_cast<Real *>(Fl + size_t(NP) * NT * sizeof(Pr<Real>));
        rho_own = Real(1) + m[0];
        {
            Real A[Basis<LAT, REC>::NH];
            // product form in fp64 only: in fp32 the factors E(c) = w(c) + O(u) round
            // their small part against the O(1) weight (1000-step parity error
            // u 7.2e-5 vs 1.9e-5 for the sum-factorised form, profiles/r03/probe.txt)
            if constexpr (LAT == LAT_D3Q27 && REC && Q27_PRODUCT && sizeof(Real) == 8) {
                (void)A;
                collide_reconstruct_q27r<Real>(m, omega, f0, fp);
            } else {
                if constexpr (LAT == LAT_D3Q19) collide_u36<REC, Real>(m, omega, A);
                else if constexpr (LAT == LAT_D3Q27 && REC) collide_q27r<Real>(m, omega, A);
                else collide_coeffs<LAT, REC, Real>(m, omega, A);
                reconstruct_pairs<LAT, REC, Real>(A, f0, fp);
            }
        }
        // publish the c_b != 0 movers
        if constexpr (SPLIT) {
            if (it >= 2) mbar_wait(&xempty[it & 1], ((it - 2) >> 1) & 1); // plane read out two layers ago
        }
        static_for<0, 6>([&](auto jk) AI {
            constexpr int ca = decltype(jk)::value % 3 - 1, cb = decltype(jk)::value / 3 == 0 ? -1 : 1;
            constexpr int ps = SL::pslot(ca, cb), zs = SL::zslot(ca, cb);
            if constexpr (ps >= 0) Fp[ps * NT + tid] = fp[ca + 1][cb + 1];
            if constexpr (zs >= 0) Fz[zs * NT + tid] = f0[ca + 1][cb + 1];
        });
    };
    // the exchange barrier after layer it was published (and the TMA refill of its stage)
    auto sync_layer = [&](const int it) AI {
        const int s = it % S;
        const int c = cfirst + it;
        if constexpr (SPLIT) {
            __syncwarp();
            if (tx == 0) {
                mbar_arrive(&xfull[it & 1]);
                if (!rowlane) mbar_arrive(&xempty[it & 1]); // halo rows never read the plane
            }
            // the TMA issuer (a halo-row thread) refills stage s once every warp
            // has published this layer, i.e. has read stage s
            if (tid == 0 && it + S < nl) {
                mbar_wait(&xfull[it & 1], (it >> 1) & 1);
                mbar_expect_tx(&full[s], stage_bytes);
                tma_load_4d(stage + s * SM::stage_elems, &tmap, &full[s], boxA, b0 + p.padB, 0, plane_of(c + S));
            }
            if (rowlane) mbar_wait(&xfull[it & 1], (it >> 1) & 1);
        } else {
            __syncthreads();
            if (tid == 0 && it + S < nl) {
                mbar_expect_tx(&full[s], stage_bytes);
                tma_load_4d(stage + s * SM::stage_elems, &tmap, &full[s], boxA, b0 + p.padB, 0, plane_of(c + S));
            }
        }

    };
    // consume(it): pull layer it from plane it & 1 into the accumulators (X: layer
    // it - 1, completed and stored; Y: layer it; Z: layer it + 1, started)
    auto consume = [&](const int it, Real (&Xa)[M], Real (&Ya)[M], Real (&Za)[M], const Real (&f0)[3][3],
                       const Pr<Real> (&fp)[3][3], const Real rho_own) AI {
        const int c = cfirst + it;
        const unsigned char *Fl = planes + (it & 1) * SM::plane_bytes;
        const Pr<Real> *Fp = reinterpret_cast<const Pr<Real> *>(Fl);
        const Real *Fz = reinterpret_cast<const Real *>(Fl + size_t(NP) * NT * sizeof(Pr<Real>));
        if (rowlane) {
            const int bbC = (c == 0 && wallClo) ? -1 : ((c == nC - 1 && wallChi) ? 1 : 0);
            auto body = [&](auto open_tag) AI {
                constexpr bool OPEN = decltype(open_tag)::value;
                auto wt = [&](int kx, int ky) AI -> Real {
                    const int cn = kx * nx_in + ky * ny_in;
                    return cn > 0 ? Real(0) : (cn < 0 ? Real(2) : Real(1));
                };
                // pairs (c_m = -1, +1): arrivals from (a - ca, b - cb)
                auto Gp = [&](auto iac, auto ibc) AI {
                    constexpr int ca = decltype(iac)::value - 1, cb = decltype(ibc)::value - 1;
                    if constexpr (dir_of<L>(ca, cb, 1) < 0) {
                        return OV<false, Pr<Real>>{};
                    } else {
                        Pr<Real> v;
                        if constexpr (cb != 0) v = Fp[SL::pslot(ca, cb) * NT + (ty - cb) * TA + (tx - ca)];
                        else if constexpr (ca != 0)
                            v = mkpr(__shfl_sync(0xffffffffu, fp[ca + 1][1].lo(), tx - ca),
                                     __shfl_sync(0xffffffffu, fp[ca + 1][1].hi(), tx - ca));
                        else v = fp[1][1];
                        if constexpr (OPEN) v = vmul(wt(ca, cb), v);
                        return OV<true, Pr<Real>>{v};
                    }
                };
                auto G0 = [&](auto iac, auto ibc) AI {
                    constexpr int ca = decltype(iac)::value - 1, cb = decltype(ibc)::value - 1;
                    if constexpr (dir_of<L>(ca, cb, 0) < 0) {
                        return OV<false, Real>{};
                    } else {
                        Real v;
                        if constexpr (cb != 0) v = Fz[SL::zslot(ca, cb) * NT + (ty - cb) * TA + (tx - ca)];
                        else if constexpr (ca != 0) v = __shfl_sync(0xffffffffu, f0[ca + 1][1], tx - ca);
                        else v = f0[1][1];
                        if constexpr (OPEN) v *= wt(ca, cb);
                        return OV<true, Real>{v};
                    }
                };
                // c_m = -1 completes layer c-1, c_m = +1 starts layer c+1
                const auto cp = colsums(Gp);
                acc_cols<-1, false, Real>(Xa, cols_half<false>(cp));
                if (c - 1 >= c0 && c - 1 < c1) finalize_store(Xa, c - 1);
                acc_cols<1, true, Real>(Za, cols_half<true>(cp));
                acc_cols<0, false, Real>(Ya, colsums(G0));
                // halfway bounce-back at walls (R12, R13), out of line
                if (bbA | bbB | bbC) {
                    auto popk = [&](auto kk) AI -> Real {
                        constexpr int k = decltype(kk)::value;
                        constexpr int ca = X::ca(k), cb = X::cb(k), cm = X::cm(k);
                        if constexpr (cb != 0) {
                            if constexpr (cm == 0) return Fz[SL::zslot(ca, cb) * NT + tid];
                            else {
                                const Pr<Real> v = Fp[SL::pslot(ca, cb) * NT + tid];
                                return cm < 0 ? v.lo() : v.hi();
                            }
                        } else {
                            if constexpr (cm == 0) return f0[ca + 1][1];
                            else return cm < 0 ? fp[ca + 1][1].lo() : fp[ca + 1][1].hi();
                        }
                    };
                    Real fk[L::Q];
                    static_for<0, L::Q>([&](auto kk) AI { fk[decltype(kk)::value] = popk(kk); });
                    const RVec<Real, M> d = bounce_back<LAT, Real, 0, false>(nullptr, fk, bbA, bbB, bbC, rho_own, &p,
                                                                              nx_in, ny_in, OPEN);
#pragma unroll
                    for (int q = 0; q < M; q++) Ya[q] += d.v[q];
                }
            };
            if (cta_open) body(std::true_type{});
            else body(std::false_type{});
            if constexpr (SPLIT) {
                __syncwarp();
                if (tx == 0) mbar_arrive(&xempty[it & 1]); // done reading this plane
            }
        }
    };
    auto layer = [&](const int it, Real (&Xa)[M], Real (&Ya)[M], Real (&Za)[M]) AI {
        Real f0[3][3];
        Pr<Real> fp[3][3];
        Real rho_own;
        produce(it, f0, fp, rho_own);
        sync_layer(it);
        consume(it, Xa, Ya, Za, f0, fp, rho_own);
    };
    // two accumulator sets with alternating roles (sweep unrolled by two, no
    // accumulator moves) wherever it fits the register file without spills: all
    // but D3Q27 recursive fp64, which keeps three rotating sets
    // ONEBODY: one layer body and three rotating sets (half the loop code: the
    // instruction-cache footprint of the sweep, at 2 M register moves per layer)
    // ROTATE: the barrier closes each iteration and the block between two barriers
    // holds the pulls of layer it and the collision + reconstruction of layer
    // it + 1 -- independent work the compiler interleaves (the FMA-bound synthesis
    // of one layer overlaps the LSU-bound pulls of the other inside each warp).
    // Plane it & 1 is read by consume(it) and next written by produce(it + 2),
    // two barriers later; stage it % S is read by produce(it) before sync_layer(it).
    if constexpr (ROTATE && !SPLIT && !ONEBODY && !(LAT == LAT_D3Q27 && REC && sizeof(Real) == 8)) {
        Real f0A[3][3], f0B[3][3];
        Pr<Real> fpA[3][3], fpB[3][3];
        Real rA, rB;
        produce(0, f0A, fpA, rA);
        sync_layer(0);
        for (int it = 0; it < nl; it += 2) {
            if (it + 1 < nl) produce(it + 1, f0B, fpB, rB);
            consume(it, accA, accB, accA, f0A, fpA, rA);
            if (it + 1 < nl) {
                sync_layer(it + 1);
                if (it + 2 < nl) produce(it + 2, f0A, fpA, rA);
                consume(it + 1, accB, accA, accB, f0B, fpB, rB);
                if (it + 2 < nl) sync_layer(it + 2);
            }
        }
        if (owner && clast == c1 - 1) {
            if (nl & 1) finalize_store(accB, c1 - 1);
            else finalize_store(accA, c1 - 1);
        }
    } else if constexpr (!ONEBODY && !(LAT == LAT_D3Q27 && REC && sizeof(Real) == 8)) {
        for (int it = 0; it < nl; it += 2) {
            layer(it, accA, accB, accA);
            if (it + 1 < nl) layer(it + 1, accB, accA, accB);
        }
        if (owner && clast == c1 - 1) {
            if (nl & 1) finalize_store(accB, c1 - 1);
            else finalize_store(accA, c1 - 1);
        }
    } else {
        for (int it = 0; it < nl; it++) {
            layer(it, accA, accB, accC);
#pragma unroll
            for (int q = 0; q < M; q++) {
                accA[q] = accB[q];
                accB[q] = accC[q];
            }
        }
        if (owner && clast == c1 - 1) finalize_store(accA, c1 - 1);
    }
}

#undef AI

} // namespace mr
