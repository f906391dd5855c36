// lattice.cuh -- compile-time lattice and Hermite-basis tables of the CUDA path.
//
// Written independently of oracle/ (which has its own tables): the standard
// single-speed lattices (Qian et al. [10]; reading R1, c_s^2 = 1/3) in
// the velocity ordering documented in include/mrlbm.h, and the Hermite
// components retained per lattice and regularization (R10):
//   projective: orders <= 2 (eq 11)
//   recursive : + the eq-14 higher orders: D2Q9 {0,1,2}^2,
//               D3Q19 (2,1,0)- and (2,2,0)-permutations, D3Q27 {0,1,2}^3.
// Every table is constexpr so that, once the per-direction loops are unrolled
// with static_for, each velocity component / weight / Hermite value is an
// immediate in the SASS.
#pragma once
#include <type_traits>
#include <utility>

namespace mr {

template <int I, int N, class F>
__device__ __forceinline__ void static_for(F &&f)
{
    if constexpr (I < N) {
        f(std::integral_constant<int, I>{});
        static_for<I + 1, N>(f);
    }
}

enum { LAT_D2Q9 = 0, LAT_D3Q19 = 1, LAT_D3Q27 = 2 };

template <int LAT> struct Lattice;

template <> struct Lattice<LAT_D2Q9> {
    static constexpr int D = 2, Q = 9, HALF = 4, M = 6;
    static constexpr int c[9][3] = {{0, 0, 0},  {1, 0, 0},  {0, 1, 0},   {1, 1, 0},  {1, -1, 0},
                                    {-1, 0, 0}, {0, -1, 0}, {-1, -1, 0}, {-1, 1, 0}};
    static constexpr double w[9] = {4.0 / 9,  1.0 / 9, 1.0 / 9,  1.0 / 36, 1.0 / 36,
                                    1.0 / 9,  1.0 / 9, 1.0 / 36, 1.0 / 36};
};

template <> struct Lattice<LAT_D3Q19> {
    static constexpr int D = 3, Q = 19, HALF = 9, M = 10;
    static constexpr int c[19][3] = {
        {0, 0, 0},  {1, 0, 0},  {0, 1, 0},  {0, 0, 1},   {1, 1, 0},  {1, -1, 0}, {1, 0, 1},
        {1, 0, -1}, {0, 1, 1},  {0, 1, -1}, {-1, 0, 0},  {0, -1, 0}, {0, 0, -1}, {-1, -1, 0},
        {-1, 1, 0}, {-1, 0, -1}, {-1, 0, 1}, {0, -1, -1}, {0, -1, 1}};
    static constexpr double w[19] = {1.0 / 3,  1.0 / 18, 1.0 / 18, 1.0 / 18, 1.0 / 36,
                                     1.0 / 36, 1.0 / 36, 1.0 / 36, 1.0 / 36, 1.0 / 36,
                                     1.0 / 18, 1.0 / 18, 1.0 / 18, 1.0 / 36, 1.0 / 36,
                                     1.0 / 36, 1.0 / 36, 1.0 / 36, 1.0 / 36};
};

template <> struct Lattice<LAT_D3Q27> {
    static constexpr int D = 3, Q = 27, HALF = 13, M = 10;
    static constexpr int c[27][3] = {
        {0, 0, 0},    {1, 0, 0},   {0, 1, 0},   {0, 0, 1},    {1, 1, 0},   {1, -1, 0},  {1, 0, 1},
        {1, 0, -1},   {0, 1, 1},   {0, 1, -1},  {1, 1, 1},    {1, 1, -1},  {1, -1, 1},  {1, -1, -1},
        {-1, 0, 0},   {0, -1, 0},  {0, 0, -1},  {-1, -1, 0},  {-1, 1, 0},  {-1, 0, -1}, {-1, 0, 1},
        {0, -1, -1},  {0, -1, 1},  {-1, -1, -1}, {-1, -1, 1}, {-1, 1, -1}, {-1, 1, 1}};
    static constexpr double w[27] = {
        8.0 / 27,  2.0 / 27,  2.0 / 27,  2.0 / 27,  1.0 / 54,  1.0 / 54,  1.0 / 54,
        1.0 / 54,  1.0 / 54,  1.0 / 54,  1.0 / 216, 1.0 / 216, 1.0 / 216, 1.0 / 216,
        2.0 / 27,  2.0 / 27,  2.0 / 27,  1.0 / 54,  1.0 / 54,  1.0 / 54,  1.0 / 54,
        1.0 / 54,  1.0 / 54,  1.0 / 216, 1.0 / 216, 1.0 / 216, 1.0 / 216};
};

// Hermite components (a,b,c): He_a(c_x) He_b(c_y) He_c(c_z).
template <int LAT, bool REC> struct Basis;

template <> struct Basis<LAT_D2Q9, false> {
    static constexpr int NH = 6;
    static constexpr int h[6][3] = {{0, 0, 0}, {1, 0, 0}, {0, 1, 0}, {2, 0, 0}, {0, 2, 0}, {1, 1, 0}};
};
template <> struct Basis<LAT_D2Q9, true> {
    static constexpr int NH = 9;
    static constexpr int h[9][3] = {{0, 0, 0}, {1, 0, 0}, {0, 1, 0}, {2, 0, 0}, {0, 2, 0},
                                    {1, 1, 0}, {2, 1, 0}, {1, 2, 0}, {2, 2, 0}};
};

#define MR_BASIS3_P                                                                              \
    {0, 0, 0}, {1, 0, 0}, {0, 1, 0}, {0, 0, 1}, {2, 0, 0}, {0, 2, 0}, {0, 0, 2}, {1, 1, 0},       \
        {1, 0, 1}, {0, 1, 1}

template <> struct Basis<LAT_D3Q19, false> {
    static constexpr int NH = 10;
    static constexpr int h[10][3] = {MR_BASIS3_P};
};
template <> struct Basis<LAT_D3Q27, false> {
    static constexpr int NH = 10;
    static constexpr int h[10][3] = {MR_BASIS3_P};
};
template <> struct Basis<LAT_D3Q19, true> {
    static constexpr int NH = 19;
    static constexpr int h[19][3] = {MR_BASIS3_P, {2, 1, 0}, {2, 0, 1}, {1, 2, 0}, {0, 2, 1}, {1, 0, 2},
                                     {0, 1, 2},   {2, 2, 0}, {2, 0, 2}, {0, 2, 2}};
};
template <> struct Basis<LAT_D3Q27, true> {
    static constexpr int NH = 27;
    static constexpr int h[27][3] = {MR_BASIS3_P, {2, 1, 0}, {2, 0, 1}, {1, 2, 0}, {0, 2, 1},
                                     {1, 0, 2},   {0, 1, 2}, {1, 1, 1}, {2, 2, 0}, {2, 0, 2},
                                     {0, 2, 2},   {2, 1, 1}, {1, 2, 1}, {1, 1, 2}, {2, 2, 1},
                                     {2, 1, 2},   {1, 2, 2}, {2, 2, 2}};
};
#undef MR_BASIS3_P

// ---- compile-time helpers -------------------------------------------------
constexpr int hfact(int k) { return k == 2 ? 2 : 1; }
constexpr int ipow3(int n) { return n == 0 ? 1 : 3 * ipow3(n - 1); }

// Scaled Hermite value He'_k(c): He'_0 = 1, He'_1 = c, He'_2 = 3c^2 - 1
// (= 3 He_2 with c_s^2 = 1/3, so every value is a small integer).
constexpr int he1s(int k, int c) { return k == 0 ? 1 : (k == 1 ? c : 3 * c * c - 1); }

// Per-component reconstruction scale 1/(a!b!c! c_s^{2n}) / 3^{#2s}  (R9), which
// pairs with He'; e.g. (2,0,0): 3/2, (1,1,0): 9, (2,1,0): 9/2, (2,2,2): 27/8.
constexpr double hscale(int a, int b, int c)
{
    int n = a + b + c;
    int n2 = (a == 2) + (b == 2) + (c == 2);
    return double(ipow3(n)) / double(hfact(a) * hfact(b) * hfact(c)) / double(ipow3(n2));
}

// slot of a moment / accumulator: 0 rho, 1+a velocity, then Pi (ABI order)
template <int D> constexpr int pslot(int a, int b)
{
    if (a > b) { int t = a; a = b; b = t; }
    if (D == 2) return a == b ? 3 + a : 5;
    if (a == b) return 4 + a;
    return a == 0 ? (b == 1 ? 7 : 8) : 9;
}

// Kernel axes: A = x (fast, in-plane), B = y (3D in-plane; absent in 2D),
// C = the marching axis (z in 3D, y in 2D) along which a CTA sweeps layers.
template <class L> struct Axes {
    static constexpr int ca(int i) { return L::c[i][0]; }
    static constexpr int cb(int i) { return L::D == 3 ? L::c[i][1] : 0; }
    static constexpr int cm(int i) { return L::D == 3 ? L::c[i][2] : L::c[i][1]; }
    static constexpr bool moving(int i) { return ca(i) != 0 || cb(i) != 0; }
    static constexpr int slot(int i)
    {
        int s = 0;
        for (int k = 0; k < i; k++) s += moving(k) ? 1 : 0;
        return s;
    }
    static constexpr int NMOVE = slot(L::Q);
    // movers along B (c_b != 0): the ones that cross warps when a warp holds one
    // A-row of the tile (3D kernels); the others move along A only
    static constexpr bool bmover(int i) { return cb(i) != 0; }
    static constexpr int bslot(int i)
    {
        int s = 0;
        for (int k = 0; k < i; k++) s += bmover(k) ? 1 : 0;
        return s;
    }
    static constexpr int NBMOVE = bslot(L::Q);
    static constexpr int opp(int i) { return i == 0 ? 0 : (i <= L::HALF ? i + L::HALF : i - L::HALF); }
};

} // namespace mr
