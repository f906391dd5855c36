// var_d3q27.cu -- the D3Q27 instances of the fused step kernel and its side kernels.
#include "var_tiles.cuh"

namespace mrd {

Variant pick_d3q27(bool rec, bool f32, int tile, int cluster)
{
    if (rec) return f32 ? pick<mr::LAT_D3Q27, true, float>(tile, cluster) : pick<mr::LAT_D3Q27, true, double>(tile, cluster);
    return f32 ? pick<mr::LAT_D3Q27, false, float>(tile, cluster) : pick<mr::LAT_D3Q27, false, double>(tile, cluster);
}

} // namespace mrd
