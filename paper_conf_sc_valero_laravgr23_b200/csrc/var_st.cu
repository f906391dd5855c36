// var_st.cu -- the distribution-representation (ST, Alg. 1) instances.
#include "dispatch.cuh"

namespace mrd {

template <int LAT> StVariant pick_st(int coll, bool f32)
{
    if (coll == MRLBM_BGK) return f32 ? make_st<LAT, mr::COLL_BGK, float>() : make_st<LAT, mr::COLL_BGK, double>();
    if (coll == MRLBM_RECURSIVE)
        return f32 ? make_st<LAT, mr::COLL_RECURSIVE, float>() : make_st<LAT, mr::COLL_RECURSIVE, double>();
    return f32 ? make_st<LAT, mr::COLL_PROJECTIVE, float>() : make_st<LAT, mr::COLL_PROJECTIVE, double>();
}

StVariant select_st(int lat, int coll, int prec)
{
    const bool F = prec == MRLBM_FP32;
    if (lat == MRLBM_D2Q9) return pick_st<mr::LAT_D2Q9>(coll, F);
    if (lat == MRLBM_D3Q19) return pick_st<mr::LAT_D3Q19>(coll, F);
    return pick_st<mr::LAT_D3Q27>(coll, F);
}


void moments_of_populations(int lat, double *pops, double *mom, int nx, int rows, cudaStream_t st)
{
    // a dense [Q][rows][nx] view; the ST set kernel stores the shifted
    // populations in place, the ST moment kernel reads them back
    mr::StGrid g;
    g.nx = nx;
    g.ny = rows;
    g.nz = 1;
    g.pitch = nx;
    g.plane = (long long)rows * nx;
    g.qstride = g.plane;
    const long long N = g.plane;
    if (lat == MRLBM_D2Q9) {
        mr::st_set_populations_kernel<mr::LAT_D2Q9, double><<<grid_for(N), 256, 0, st>>>(pops, pops, g);
        mr::st_get_moments_kernel<mr::LAT_D2Q9, double><<<grid_for(N), 256, 0, st>>>(pops, mom, g);
    } else if (lat == MRLBM_D3Q19) {
        mr::st_set_populations_kernel<mr::LAT_D3Q19, double><<<grid_for(N), 256, 0, st>>>(pops, pops, g);
        mr::st_get_moments_kernel<mr::LAT_D3Q19, double><<<grid_for(N), 256, 0, st>>>(pops, mom, g);
    } else {
        mr::st_set_populations_kernel<mr::LAT_D3Q27, double><<<grid_for(N), 256, 0, st>>>(pops, pops, g);
        mr::st_get_moments_kernel<mr::LAT_D3Q27, double><<<grid_for(N), 256, 0, st>>>(pops, mom, g);
    }
}

} // namespace mrd
