// var_d3q19.cu -- the D3Q19 instances of the fused step kernel and its side kernels.
#include "var_tiles.cuh"

namespace mrd {

Variant pick_d3q19(bool rec, bool f32, int tile)
{
    if (rec) return f32 ? pick<mr::LAT_D3Q19, true, float>(tile) : pick<mr::LAT_D3Q19, true, double>(tile);
    return f32 ? pick<mr::LAT_D3Q19, false, float>(tile) : pick<mr::LAT_D3Q19, false, double>(tile);
}

} // namespace mrd
