// var_d3q19.cu -- the D3Q19 instances of the fused step kernel and its side kernels.
#include "var_tiles.cuh"

namespace mrd {

Variant pick_d3q19(bool rec, bool f32, int tile, int cluster)
{
    if (rec) return f32 ? pick<mr::LAT_D3Q19, true, float>(tile, cluster) : pick<mr::LAT_D3Q19, true, double>(tile, cluster);
    return f32 ? pick<mr::LAT_D3Q19, false, float>(tile, cluster) : pick<mr::LAT_D3Q19, false, double>(tile, cluster);
}

} // namespace mrd
