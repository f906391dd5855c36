// var_tiles.cuh -- tile shapes per lattice; included by
// the per-lattice translation units only.
#pragma once
#include "dispatch.cuh"

namespace mrd {

// 3D default: clusters of two CTAs along B (see mrlbm_step_kernel, CL)
constexpr bool kClusterDefault = false;

// Tile shapes: 2D one row of 128 threads (126 interior
// nodes); 3D either 32 x 8 threads (30 x 6 interior, 2 CTAs/SM) or 32 x 16
// threads (30 x 14 interior, 1 CTA/SM).  tile = 0: library default, 1: 32x8,
// 2: 32x16 (MRLBM_TILE overrides, for tuning).
template <int LAT, bool REC, typename Real> Variant pick(int tile, int cluster)
{
    if constexpr (LAT == mr::LAT_D2Q9) {
        (void)cluster;
        // deeper TMA rings trade resident CTAs for bytes in flight (tuning: MRLBM_TILE)
        // (the round-2 ring-depth sweep variants 2..7 are retired: profiles/ring2d_*_r02.jsonl)
        if (tile == 1) return make_variant<LAT, REC, Real, 128, 1, 4, 4>();
        if (tile == 8) return make_variant<LAT, REC, Real, 128, 1, 4, 5>(); // round-1 default
        // default: a 6-deep TMA ring; fp64 at 4 CTAs/SM (6 x 6.2 KB stages), fp32 at 6
        // (measured C2: fp64 0.90 -> 0.916, fp32 0.80 -> 0.82; profiles/ring2d_b_r02.jsonl)
        if constexpr (sizeof(Real) == 8) return make_variant<LAT, REC, Real, 128, 1, 6, 4, true>();
        else return make_variant<LAT, REC, Real, 128, 1, 6, 6, true>();
    } else {
        constexpr bool f64 = sizeof(Real) == 8;
        // smem: S TMA stages + two exchange planes; D3Q27 fp64 only fits the small tile
        constexpr bool small_only = LAT == mr::LAT_D3Q27 && f64;
        // Defaults (tile 0), from the round-3 one-box A/Bs (profiles/r03/):
        //  D3Q19 fp64: the scalar kernel (mrlbm_step_kernel, 32 x 8, 2 CTAs/SM) with
        //         the regrouped collision -- the paired kernel's fp64 pair registers
        //         cost moves (+8% instructions on C3) and it measured 1-5% slower;
        //  D3Q19 fp32 and D3Q27: the paired kernel (step3d.cuh) on 32 x 8 tiles at
        //         2 CTAs/SM (packed FP32; C3 fp32 +3%, C4 fp32 +4% over the scalar
        //         kernel; C4 fp64 +14% with the product-form D3Q27-R).
        // tile 9 selects the round-2 default shapes of the scalar kernel (A/B).
        if (tile == 0 && cluster != 2) {
            if constexpr (LAT == mr::LAT_D3Q27 || !f64) return make_variant3<LAT, REC, Real, 8, 3, 2, true>();
        }
        // tile 15: the paired kernel on the 32 x 16 tile (one CTA per SM)
        if (tile == 15) {
            if constexpr (!small_only) return make_variant3<LAT, REC, Real, 16, (f64 ? 2 : 4), 1, true>();
        }
        // tile 10: the paired kernel on 32 x 8 tiles at 2 CTAs/SM (A/B for D3Q27 fp32)
        if (tile == 10) {
            if constexpr (!small_only) return make_variant3<LAT, REC, Real, 8, 3, 2, true>();
        }
        // (round-3 A/B variants retired after measurement, profiles/r03/: tile 11/12
        // split-phase barriers, 13/14 one-body sweeps, 16 a 5-deep paired ring; the
        // kernel keeps the SPLIT / ONEBODY template options)
        if (tile == 9) tile = 0;
        const bool dflt = tile == 0;
        if (tile == 0) tile = (LAT == mr::LAT_D3Q19 || small_only) ? 1 : 2;
        // TMA ring depth: with the A-movers exchanged by shuffles the fp64 32x8
        // tile fits three stages at two CTAs per SM; the 32x16 tile (one CTA
        // per SM) takes four in fp32
        // the library defaults also carry the P2P push instance
        constexpr bool small_default = LAT == mr::LAT_D3Q19 || small_only;
        // clusters of 2 CTAs along B (DSMEM mover exchange, no halo rows between
        // them): cluster = 0 library default, 1 off, 2 on (MRLBM_CLUSTER)
        const bool cl2 = dflt && (cluster == 2 || (cluster == 0 && kClusterDefault));
        if constexpr (!f64) { // fp32 32x16: deeper TMA ring (tuning: MRLBM_TILE=3)
            if (tile == 3) return make_variant<LAT, REC, Real, 32, 16, 6, 1>();
        }
        if (tile == 1 || small_only) {
            if (cl2) return make_variant<LAT, REC, Real, 32, 8, 3, 2, small_default, 2>();
            return make_variant<LAT, REC, Real, 32, 8, 3, 2, small_default>();
        }
        if (cl2) return make_variant<LAT, REC, Real, 32, 16, (f64 ? 2 : 4), 1, !small_default, 2>();
        return make_variant<LAT, REC, Real, 32, 16, (f64 ? 2 : 4), 1, !small_default>();
    }
}

} // namespace mrd
