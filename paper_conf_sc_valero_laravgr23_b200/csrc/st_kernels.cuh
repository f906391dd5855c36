// st_kernels.cuh -- the standard DISTRIBUTION representation (ST) on sm_100a:
// the paper's comparison baseline (Alg. 1).
//
// The state is the Q pre-collision populations per node in two lattices
// ("we need two different lattices ... to compute the streaming stage
// in parallel"), structure-of-arrays [q][z][y][x] (P:L189 SoA, coalesced).
// One launch = one timestep: each thread reads its node's Q populations
// (coalesced), collides (BGK = Alg. 1 lines 21-25; or the projective /
// recursive regularized operators of the MR path, eqs 9-14, computed in
// distribution form from the node's moments) and pushes the post-collision
// populations to x + c_i in the other lattice (eq 7).  Walls: halfway
// bounce-back with the Ladd moving-wall term (R12, R13), exactly as the
// oracle.  Bytes per lattice update: 2 Q w (Table 2).
//
// Why push and not the paper's pull: on V100 uncoalesced stores cost
// more than uncoalesced loads.  On B200 a store shifted by one element is
// merged in L2 before write-back, and push keeps the state pre-collision, so
// get_moments needs no gather and the boundary rule is the oracle's own.
// Like the MR path the state is stored shifted (f - w_i, R16).
#pragma once
#include "mrlbm_kernels.cuh"

namespace mr {

struct StArgs {
    const void *src;
    void *dst;
    int nx, ny, nz, pitch;
    long long plane;   // ny * pitch
    long long qstride; // nz * plane
    int kind[6];       // physical faces x-, x+, y-, y+, z-, z+ (2D: z faces periodic)
    double uw[6][3];   // moving-wall velocities
    double omega;      // 1 - 1/tau
    double inv_tau;    // 1/tau
};

enum { COLL_PROJECTIVE = 0, COLL_RECURSIVE = 1, COLL_BGK = 2 };

// Raw moments of shifted populations: S0 = sum f~ (= rho - 1), j = sum c f~
// (= rho u), and Pi (eq 3) = sum c c f~ - c_s^2 delta S0.
template <int LAT, typename Real>
__device__ __forceinline__ void st_moments(const Real (&f)[Lattice<LAT>::Q], Real (&m)[Lattice<LAT>::M], Real &S0,
                                           Real (&j)[3])
{
    using L = Lattice<LAT>;
    constexpr int D = L::D, M = L::M;
    Real s[M];
#pragma unroll
    for (int q = 0; q < M; q++) s[q] = Real(0);
    static_for<0, L::Q>([&](auto kk) {
        constexpr int k = decltype(kk)::value;
        s[0] += f[k];
        static_for<0, D>([&](auto ak) {
            constexpr int a = decltype(ak)::value;
            acc_int<L::c[k][a]>(s[1 + a], f[k]);
            static_for<a, D>([&](auto bk) {
                constexpr int b = decltype(bk)::value;
                acc_int<L::c[k][a] * L::c[k][b]>(s[pslot<D>(a, b)], f[k]);
            });
        });
    });
    S0 = s[0];
    const Real inv = rcp_nr(Real(1) + S0);
    m[0] = S0;
    j[2] = Real(0);
#pragma unroll
    for (int a = 0; a < D; a++) {
        j[a] = s[1 + a];
        m[1 + a] = s[1 + a] * inv;
    }
#pragma unroll
    for (int a = 0; a < D; a++)
#pragma unroll
        for (int b = a; b < D; b++) m[pslot<D>(a, b)] = s[pslot<D>(a, b)] - ((a == b) ? S0 * Real(1.0 / 3.0) : Real(0));
}

// Post-collision shifted populations of one node from its pre-collision ones.
template <int LAT, int COLL, typename Real>
__device__ __forceinline__ void st_collide(const Real (&f)[Lattice<LAT>::Q], Real (&fs)[Lattice<LAT>::Q], Real omega,
                                           Real inv_tau, Real &rho_out)
{
    using L = Lattice<LAT>;
    constexpr int D = L::D;
    Real m[L::M], S0, j[3];
    st_moments<LAT, Real>(f, m, S0, j);
    const Real rho = Real(1) + S0;
    rho_out = rho;
    if constexpr (COLL == COLL_BGK) {
        // Alg. 1 lines 21-25 with eq 4 (R2), shifted: f~eq_i = w_i (S0 + rho (3cu + 9/2 cu^2 - 3/2 u^2))
        Real u[3] = {m[1], m[2], D == 3 ? m[3] : Real(0)};
        const Real usq = u[0] * u[0] + u[1] * u[1] + u[2] * u[2];
        const Real base = fma(Real(-1.5) * rho, usq, S0);
        const Real r3 = Real(3) * rho, r45 = Real(4.5) * rho;
        static_for<0, L::HALF + 1>([&](auto ik) {
            constexpr int i = decltype(ik)::value;
            constexpr Real w = Real(L::w[i]);
            Real cu = Real(0);
            static_for<0, D>([&](auto ak) {
                constexpr int a = decltype(ak)::value;
                acc_int<L::c[i][a]>(cu, u[a]);
            });
            const Real E = fma(r45 * cu, cu, base);
            const Real O = r3 * cu;
            fs[i] = fma(omega, f[i], inv_tau * (w * (E + O)));
            if constexpr (i > 0) fs[i + L::HALF] = fma(omega, f[i + L::HALF], inv_tau * (w * (E - O)));
        });
    } else {
        constexpr bool REC = COLL == COLL_RECURSIVE;
        Real A[Basis<LAT, REC>::NH];
        collide_coeffs<LAT, REC, Real>(m, omega, A);
        reconstruct<LAT, REC, Real>(A, fs);
    }
}

// Push of the post-collision populations of a node on the domain boundary
// (oracle step 4): wrap periodic axes; a population leaving through a wall
// returns to its own node as opp(i), minus 2 w_i rho (c_i.u_w)/c_s^2 for every
// moving wall crossed (R12, R13).  Only boundary nodes run it; inlined so that
// the populations stay in registers (an out-of-line call taking them by
// pointer put every thread's populations on the stack: +2.4 GB of local
// stores per C3 step, measured).
template <int LAT, typename Real>
__device__ __forceinline__ void st_store_boundary(const Real (&fs)[Lattice<LAT>::Q], Real rho, Real *dst, int x, int y,
                                                  int z, const StArgs *p)
{
    using L = Lattice<LAT>;
    using X = Axes<L>;
    const int n[3] = {p->nx, p->ny, p->nz};
    const long long own = (long long)z * p->plane + (long long)y * p->pitch + x;
    static_for<0, L::Q>([&](auto kk) {
        constexpr int k = decltype(kk)::value;
        constexpr int cx = L::c[k][0], cy = L::c[k][1], cz = L::c[k][2];
        int d[3] = {x + cx, y + cy, z + cz};
        bool wall = false;
        double cuw = 0.0;
#pragma unroll
        for (int a = 0; a < 3; a++) {
            if (d[a] >= 0 && d[a] < n[a]) continue;
            const int face = 2 * a + (d[a] < 0 ? 0 : 1);
            if (p->kind[face] == BC_PERIODIC) {
                d[a] = d[a] < 0 ? d[a] + n[a] : d[a] - n[a];
            } else {
                wall = true;
                if (p->kind[face] == BC_MOVING)
                    cuw += cx * p->uw[face][0] + cy * p->uw[face][1] + cz * p->uw[face][2];
            }
        }
        if (wall) {
            constexpr int ko = X::opp(k);
            constexpr double wk6 = 6.0 * L::w[k];
            dst[ko * p->qstride + own] = fs[k] - Real(wk6) * rho * Real(cuw);
        } else {
            dst[k * p->qstride + (long long)d[2] * p->plane + (long long)d[1] * p->pitch + d[0]] = fs[k];
        }
    });
}

template <int LAT, int COLL, typename Real, int BX>
__global__ void __launch_bounds__(BX, 4) st_step_kernel(const StArgs p)
{
    using L = Lattice<LAT>;
    constexpr int Q = L::Q;
    const int x = blockIdx.x * BX + threadIdx.x;
    const int y = blockIdx.y, z = blockIdx.z;
    if (x >= p.nx) return;
    const long long own = (long long)z * p.plane + (long long)y * p.pitch + x;
    const Real *src = reinterpret_cast<const Real *>(p.src) + own;
    Real *dst = reinterpret_cast<Real *>(p.dst);
    Real f[Q];
#pragma unroll
    for (int i = 0; i < Q; i++) f[i] = __ldcs(src + i * p.qstride); // streamed once: evict-first
    Real fs[Q], rho;
    st_collide<LAT, COLL, Real>(f, fs, Real(p.omega), Real(p.inv_tau), rho);
    const bool inner = x > 0 && x < p.nx - 1 && y > 0 && y < p.ny - 1 && (L::D == 2 || (z > 0 && z < p.nz - 1));
    if (inner) {
        static_for<0, Q>([&](auto kk) {
            constexpr int k = decltype(kk)::value;
            constexpr int cx = L::c[k][0], cy = L::c[k][1], cz = L::c[k][2];
            const long long off = cx + (long long)cy * p.pitch + (long long)cz * p.plane;
            dst[k * p.qstride + own + off] = fs[k];
        });
    } else {
        st_store_boundary<LAT, Real>(fs, rho, dst, x, y, z, &p);
    }
}

// ---- state I/O (fp64 ABI arrays [.][nz][ny][nx])
struct StGrid {
    int nx, ny, nz, pitch;
    long long plane, qstride;
};

__device__ __forceinline__ long long st_index(const StGrid &g, long long n, int &x)
{
    x = int(n % g.nx);
    const long long r = n / g.nx;
    const int y = int(r % g.ny), z = int(r / g.ny);
    return (long long)z * g.plane + (long long)y * g.pitch + x;
}

// moments -> regularized populations f~ = w (rho + c.rho u/c_s^2 + H2:Pi/(2 c_s^4)) - w
// (the projective reconstruction without relaxation, eq 11 with omega = 1)
template <int LAT, typename Real>
__global__ void st_set_moments_kernel(const double *__restrict__ in, Real *__restrict__ buf, StGrid g)
{
    using L = Lattice<LAT>;
    const long long N = (long long)g.nx * g.ny * g.nz;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        int x;
        const long long o = st_index(g, n, x);
        Real m[L::M];
#pragma unroll
        for (int q = 0; q < L::M; q++) m[q] = Real(in[q * N + n] - (q == 0 ? 1.0 : 0.0));
        Real A[Basis<LAT, false>::NH], f[L::Q];
        collide_coeffs<LAT, false, Real>(m, Real(1), A);
        reconstruct<LAT, false, Real>(A, f);
#pragma unroll
        for (int i = 0; i < L::Q; i++) buf[i * g.qstride + o] = f[i];
    }
}

template <int LAT, typename Real>
__global__ void st_set_populations_kernel(const double *__restrict__ in, Real *__restrict__ buf, StGrid g)
{
    using L = Lattice<LAT>;
    const long long N = (long long)g.nx * g.ny * g.nz;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        int x;
        const long long o = st_index(g, n, x);
        static_for<0, L::Q>([&](auto kk) {
            constexpr int k = decltype(kk)::value;
            constexpr double wk = L::w[k];
            buf[k * g.qstride + o] = Real(in[k * N + n] - wk);
        });
    }
}

template <int LAT, typename Real>
__global__ void st_get_moments_kernel(const Real *__restrict__ buf, double *__restrict__ out, StGrid g)
{
    using L = Lattice<LAT>;
    const long long N = (long long)g.nx * g.ny * g.nz;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        int x;
        const long long o = st_index(g, n, x);
        Real f[L::Q], m[L::M], S0, j[3];
#pragma unroll
        for (int i = 0; i < L::Q; i++) f[i] = buf[i * g.qstride + o];
        st_moments<LAT, Real>(f, m, S0, j);
#pragma unroll
        for (int q = 0; q < L::M; q++) out[q * N + n] = double(m[q]) + (q == 0 ? 1.0 : 0.0);
    }
}

// post-collision populations f* of the current state (R17), fp64 [Q][N]
template <int LAT, int COLL, typename Real>
__global__ void st_populations_kernel(const Real *__restrict__ buf, double *__restrict__ out, StGrid g, double omega,
                                      double inv_tau)
{
    using L = Lattice<LAT>;
    const long long N = (long long)g.nx * g.ny * g.nz;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        int x;
        const long long o = st_index(g, n, x);
        Real f[L::Q], fs[L::Q], rho;
#pragma unroll
        for (int i = 0; i < L::Q; i++) f[i] = buf[i * g.qstride + o];
        st_collide<LAT, COLL, Real>(f, fs, Real(omega), Real(inv_tau), rho);
        static_for<0, L::Q>([&](auto kk) {
            constexpr int k = decltype(kk)::value;
            constexpr double wk = L::w[k];
            out[k * N + n] = double(fs[k]) + wk;
        });
    }
}

template <int LAT, typename Real>
__global__ void st_finite_kernel(const Real *__restrict__ buf, StGrid g, int *flag)
{
    using L = Lattice<LAT>;
    const long long N = (long long)g.nx * g.ny * g.nz;
    for (long long n = blockIdx.x * (long long)blockDim.x + threadIdx.x; n < N; n += (long long)gridDim.x * blockDim.x) {
        int x;
        const long long o = st_index(g, n, x);
#pragma unroll
        for (int i = 0; i < L::Q; i++)
            if (!isfinite(double(buf[i * g.qstride + o]))) atomicExch(flag, 1);
    }
}

} // namespace mr
