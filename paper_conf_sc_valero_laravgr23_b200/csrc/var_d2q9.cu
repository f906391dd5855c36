// var_d2q9.cu -- the D2Q9 instances of the fused step kernel and its side kernels.
#include "var_tiles.cuh"

namespace mrd {

Variant pick_d2q9(bool rec, bool f32, int tile, int cluster)
{
    if (rec) return f32 ? pick<mr::LAT_D2Q9, true, float>(tile, cluster) : pick<mr::LAT_D2Q9, true, double>(tile, cluster);
    return f32 ? pick<mr::LAT_D2Q9, false, float>(tile, cluster) : pick<mr::LAT_D2Q9, false, double>(tile, cluster);
}

} // namespace mrd
