// var_d3q27.cu -- the D3Q27 instances of the fused step kernel and its side kernels.
#include "var_tiles.cuh"

namespace mrd {

Variant pick_d3q27(bool rec, bool f32, int tile)
{
    if (rec) return f32 ? pick<mr::LAT_D3Q27, true, float>(tile) : pick<mr::LAT_D3Q27, true, double>(tile);
    return f32 ? pick<mr::LAT_D3Q27, false, float>(tile) : pick<mr::LAT_D3Q27, false, double>(tile);
}

} // namespace mrd
