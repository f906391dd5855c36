// mrlbm.cu -- host side of libmrlbm.so: the C ABI declared in include/mrlbm.h.
//
// Owns the device state (two SoA moment buffers, ping-pong, R7), builds the
// TMA descriptors of both buffers, selects the template instance of the fused
// step kernel (lattice x regularization x precision), batches steps into
// CUDA graphs, and for nranks > 1 exchanges one boundary plane of moments per
// step with each z-slab neighbour through NCCL send/recv on a communication
// stream, overlapped with the interior update.
// With MRLBM_DISTRIBUTIONS the same handle runs the paper's standard
// distribution representation (ST, Alg. 1) instead: two Q-population lattices
// and the push kernel of st_kernels.cuh (the comparison baseline, NEXT-2).
#include <cuda.h>
#include <cuda_runtime.h>
#include <nccl.h>
#include <unistd.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

#include "../../include/mrlbm.h"
#include "dispatch.cuh"
#include "p2p_kernels.cuh"

namespace {

thread_local std::string g_last_error;

mrlbm_status fail(mrlbm_status s, const std::string &msg)
{
    g_last_error = msg;
    return s;
}

#define MR_CUDA(call)                                                                                \
    do {                                                                                            \
        cudaError_t e_ = (call);                                                                    \
        if (e_ != cudaSuccess)                                                                      \
            return fail(MRLBM_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_));        \
    } while (0)

#define MR_NCCL(call)                                                                               \
    do {                                                                                            \
        ncclResult_t r_ = (call);                                                                   \
        if (r_ != ncclSuccess) return fail(MRLBM_ERR_NCCL, std::string(#call) + ": " + ncclGetErrorString(r_)); \
    } while (0)

using mr::StepArgs;

using mrd::Variant;
using mrd::StVariant;
using mrd::select_st;
using mrd::grid_for;

Variant select_variant(int lat, int reg, int prec, int tile, int cluster)
{
    const bool R = reg == MRLBM_RECURSIVE;
    const bool F = prec == MRLBM_FP32;
    if (lat == MRLBM_D2Q9) return mrd::pick_d2q9(R, F, tile, cluster);
    if (lat == MRLBM_D3Q19) return mrd::pick_d3q19(R, F, tile, cluster);
    return mrd::pick_d3q27(R, F, tile, cluster);
}

int env_int(const char *name, int dflt)
{
    const char *v = getenv(name);
    return v && *v ? atoi(v) : dflt;
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode_fn()
{
    static EncodeTiledFn fn = nullptr;
    if (!fn) {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeTiledFn)p;
    }
    return fn;
}

} // namespace

// ---------------------------------------------------------------- context
struct mrlbm_ctx {
    int lattice, reg, prec, D, M, Q, wbytes;
    int64_t gn[3];        // global nx, ny, nz (nz = 1 in 2D)
    int nA, nB, nC;       // local kernel extents
    int cglobal, coff;    // global march extent, offset of this rank
    int pitch, padA, padB;
    long long mstride, pstride, origin; // origin: element offset of node (0,0) in a plane
    size_t buf_bytes;
    double tau, omega;
    int rank = 0, nranks = 1, device = 0;
    mrlbm_boundary bnd;   // physical faces (profiles re-pointed to device copies)
    void *buf[2] = {nullptr, nullptr};
    int cur = 0;
    CUtensorMap tmap[2];
    Variant var;
    StepArgs base;        // template of the kernel arguments (src/dst filled per launch)
    int tilesA, tilesB, seg_len, nseg;
    cudaStream_t stream = nullptr, comm_stream = nullptr, cap_stream = nullptr;
    bool own_stream = false;
    cudaEvent_t ev_ready = nullptr, ev_comm = nullptr, ev_t0 = nullptr, ev_t1 = nullptr;
    double *prof_dev[6] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
    bool fd_face[4] = {false, false, false, false}; // kernel faces A-, A+, B-, B+ with the FD scheme (R20)
    double *io = nullptr;  // fp64 staging for set/get/populations
    size_t io_bytes = 0;
    int *flag = nullptr;
    ncclComm_t comm = nullptr;
    bool group_mode = false;    // nranks > 1 without NCCL: ghosts filled by mrlbm_step_group
    // P2P transport: peer memory pushes + device counters (mrlbm_p2p_*)
    bool p2p = false, p2p_connected = false;
    unsigned long long *sync = nullptr;            // [0] own pushes, [1] from lo, [2] from hi
    int *p2p_err = nullptr;
    void *peer_plane_lo[2] = {nullptr, nullptr};   // lower neighbour's HIGH ghost plane (start), per buffer
    void *peer_plane_hi[2] = {nullptr, nullptr};   // upper neighbour's LOW ghost plane (start), per buffer
    unsigned long long *peer_sync_lo = nullptr, *peer_sync_hi = nullptr;
    std::vector<void *> ipc_opened;                // IPC mappings to close
    int nb_lo = -1, nb_hi = -1; // neighbour ranks along C (-1 none)
    cudaGraphExec_t graph[2] = {nullptr, nullptr};
    int graph_steps = 0;
    int64_t kernels = 0;
    // distribution representation (ST)
    int repr = MRLBM_MOMENTS;
    StVariant sv;
    mr::StArgs st_base;
    mr::StGrid st_grid;
};

namespace {

// pointer to node (0,0) of plane 0 of buffer i
void *node0(const mrlbm_ctx *h, int i) { return (char *)h->buf[i] + (size_t)h->origin * h->wbytes; }

mr::GridArgs grid_args(const mrlbm_ctx *h)
{
    mr::GridArgs g;
    g.nA = h->nA;
    g.nB = h->nB;
    g.nC = h->nC;
    g.pitch = h->pitch;
    g.mstride = h->mstride;
    g.pstride = h->pstride;
    g.perA = h->base.kind[0] == mr::BC_PERIODIC;
    g.perB = h->D == 3 && h->base.kind[2] == mr::BC_PERIODIC;
    return g;
}

// launch the fused kernel over owned layers [cb, ce) (and, if ce2 > cb2, also
// over [cb2, ce2) in the same launch) reading buf[src]
void launch_range(mrlbm_ctx *h, int src, int cb, int ce, cudaStream_t st, bool push = false, int cb2 = 0, int ce2 = 0)
{
    if (ce <= cb) return;
    StepArgs a = h->base;
    a.src = node0(h, src);
    a.dst = node0(h, 1 - src);
    if (push) { // P2P: layers 0 / nC-1 of the new state also go to the neighbours' ghost planes
        const size_t org = (size_t)h->origin * h->wbytes;
        a.peer_lo = h->peer_plane_lo[1 - src] ? (char *)h->peer_plane_lo[1 - src] + org : nullptr;
        a.peer_hi = h->peer_plane_hi[1 - src] ? (char *)h->peer_plane_hi[1 - src] + org : nullptr;
    }
    a.c_begin = cb;
    a.c_end = ce;
    const int span = ce - cb;
    a.seg_len = std::min(h->seg_len, span);
    a.nseg1 = (span + a.seg_len - 1) / a.seg_len;
    int nseg = a.nseg1;
    if (ce2 > cb2) { // second range: segments nseg1.. of the grid (same segment length)
        a.c2_begin = cb2;
        a.c2_end = ce2;
        nseg += (ce2 - cb2 + a.seg_len - 1) / a.seg_len;
    }
    dim3 grid(h->tilesA, h->tilesB, nseg);
    if (a.rastG > 0) grid = dim3(h->tilesA * h->tilesB, 1, nseg); // grouped launch order (kernel remaps)
    if (push) h->var.step_push(h->tmap[src], a, grid, st);
    else h->var.step(h->tmap[src], a, grid, st);
    h->kernels++;
}

// the slab's first and last layer (they read the ghost planes) in one launch
void launch_boundary(mrlbm_ctx *h, int src, cudaStream_t st, bool push)
{
    if (h->nC == 1) launch_range(h, src, 0, 1, st, push);
    else launch_range(h, src, 0, 1, st, push, h->nC - 1, h->nC);
}

mrlbm_status enqueue_one_step(mrlbm_ctx *h, cudaStream_t st)
{
    const int src = h->cur;
    if (h->repr == MRLBM_DISTRIBUTIONS) {
        mr::StArgs a = h->st_base;
        a.src = h->buf[src];
        a.dst = h->buf[1 - src];
        dim3 grid((unsigned)((h->st_grid.nx + h->sv.BX - 1) / h->sv.BX), (unsigned)h->st_grid.ny, (unsigned)h->st_grid.nz);
        h->sv.step(a, grid, st);
        h->kernels++;
    } else if (h->p2p) {
        // P2P: interior layers need no ghost plane; then wait until both
        // neighbours have pushed as often as this rank (our ghosts are current,
        // and they are done reading the ghost planes we push into), run the
        // boundary layers with the push fused into their stores, and signal
        if (!h->p2p_connected) return fail(MRLBM_ERR_INVALID_ARGUMENT, "P2P transport: mrlbm_p2p_connect first");
        launch_range(h, src, 1, h->nC - 1, st);
        mr::p2p_wait_kernel<<<1, 1, 0, st>>>(h->sync, h->nb_lo >= 0, h->nb_hi >= 0, h->p2p_err);
        launch_boundary(h, src, st, true); // layers 0 and nC-1 in one launch, pushes fused
        mr::p2p_signal_kernel<<<1, 1, 0, st>>>(h->sync, h->peer_sync_lo, h->peer_sync_hi, h->p2p_err);
        h->kernels += 2;
    } else if (h->nranks == 1) {
        launch_range(h, src, 0, h->nC, st);
        // finite-difference open faces: stress of the face nodes from the new velocity field
        for (int K = 0; K < 4; K++) {
            if (!h->fd_face[K]) continue;
            mr::FdArgs f;
            f.buf = node0(h, 1 - src);
            f.nA = h->nA;
            f.nB = h->nB;
            f.nC = h->nC;
            f.pitch = h->pitch;
            f.mstride = h->mstride;
            f.pstride = h->pstride;
            f.face = K;
            f.per[0] = h->base.kind[0] == mr::BC_PERIODIC;
            f.per[1] = h->D == 3 && h->base.kind[2] == mr::BC_PERIODIC;
            f.per[2] = h->base.wrapC;
            f.tau = h->tau;
            h->var.fd(f, (long long)(K < 2 ? h->nB : h->nA) * h->nC, st);
            h->kernels++;
        }
    } else {
        // halo exchange of the boundary planes of the current state, overlapped
        // with the interior layers [1, nC-1) that do not read the ghost planes
        MR_CUDA(cudaEventRecord(h->ev_ready, st));
        MR_CUDA(cudaStreamWaitEvent(h->comm_stream, h->ev_ready, 0));
        char *base = (char *)h->buf[src];
        const size_t plane = (size_t)h->pstride * h->wbytes;
        const ncclDataType_t dt = h->prec == MRLBM_FP32 ? ncclFloat32 : ncclFloat64;
        const size_t cnt = (size_t)h->pstride;
        MR_NCCL(ncclGroupStart());
        ncclResult_t r = ncclSuccess;
        if (r == ncclSuccess && h->nb_hi >= 0) r = ncclSend(base + plane * h->nC, cnt, dt, h->nb_hi, h->comm, h->comm_stream);
        if (r == ncclSuccess && h->nb_lo >= 0) r = ncclSend(base + plane * 1, cnt, dt, h->nb_lo, h->comm, h->comm_stream);
        if (r == ncclSuccess && h->nb_lo >= 0) r = ncclRecv(base, cnt, dt, h->nb_lo, h->comm, h->comm_stream);
        if (r == ncclSuccess && h->nb_hi >= 0)
            r = ncclRecv(base + plane * (h->nC + 1), cnt, dt, h->nb_hi, h->comm, h->comm_stream);
        const ncclResult_t re = ncclGroupEnd(); // always close the group, also on error
        if (r != ncclSuccess) return fail(MRLBM_ERR_NCCL, std::string("ncclSend/ncclRecv: ") + ncclGetErrorString(r));
        if (re != ncclSuccess) return fail(MRLBM_ERR_NCCL, std::string("ncclGroupEnd: ") + ncclGetErrorString(re));
        MR_CUDA(cudaEventRecord(h->ev_comm, h->comm_stream));
        launch_range(h, src, 1, h->nC - 1, st);
        MR_CUDA(cudaStreamWaitEvent(st, h->ev_comm, 0));
        launch_boundary(h, src, st, false); // layers 0 and nC-1 in one launch
    }
    h->cur ^= 1;
    MR_CUDA(cudaGetLastError());
    return MRLBM_OK;
}

mrlbm_status ensure_io(mrlbm_ctx *h, size_t bytes)
{
    if (h->io_bytes >= bytes) return MRLBM_OK;
    if (h->io) cudaFree(h->io);
    h->io = nullptr;
    h->io_bytes = 0;
    if (cudaMalloc(&h->io, bytes) != cudaSuccess) {
        cudaGetLastError();
        return fail(MRLBM_ERR_OUT_OF_MEMORY, "staging allocation failed");
    }
    h->io_bytes = bytes;
    return MRLBM_OK;
}

// P2P: after the state was set from outside, push its boundary planes into the
// neighbours' ghost planes of the current buffer (ordered like a step's push)
mrlbm_status p2p_prologue(mrlbm_ctx *h)
{
    if (!h->p2p) return MRLBM_OK;
    if (!h->p2p_connected) // the neighbours' ghost planes cannot be filled: refuse (header)
        return fail(MRLBM_ERR_INVALID_ARGUMENT, "P2P transport: mrlbm_p2p_connect before setting the state");
    const int b = h->cur;
    char *base = (char *)h->buf[b];
    const size_t plane = (size_t)h->pstride * h->wbytes;
    mr::p2p_wait_kernel<<<1, 1, 0, h->stream>>>(h->sync, h->nb_lo >= 0, h->nb_hi >= 0, h->p2p_err);
    if (h->prec == MRLBM_FP32)
        mr::p2p_push_planes_kernel<float><<<grid_for(h->pstride), 256, 0, h->stream>>>(
            (const float *)(base + plane), (const float *)(base + plane * h->nC), (float *)h->peer_plane_lo[b],
            (float *)h->peer_plane_hi[b], h->pstride);
    else
        mr::p2p_push_planes_kernel<double><<<grid_for(h->pstride), 256, 0, h->stream>>>(
            (const double *)(base + plane), (const double *)(base + plane * h->nC), (double *)h->peer_plane_lo[b],
            (double *)h->peer_plane_hi[b], h->pstride);
    mr::p2p_signal_kernel<<<1, 1, 0, h->stream>>>(h->sync, h->peer_sync_lo, h->peer_sync_hi, h->p2p_err);
    MR_CUDA(cudaGetLastError());
    return MRLBM_OK;
}

// P2P: a halo wait that timed out poisons the handle (its ghosts are stale)
mrlbm_status p2p_check(mrlbm_ctx *h)
{
    if (!h->p2p_err) return MRLBM_OK;
    int e = 0;
    MR_CUDA(cudaMemcpy(&e, h->p2p_err, sizeof(int), cudaMemcpyDeviceToHost));
    return e ? fail(MRLBM_ERR_CUDA, "P2P transport: a neighbour stopped (halo wait timed out)") : MRLBM_OK;
}

bool is_wall(int k) { return k == MRLBM_WALL || k == MRLBM_MOVING_WALL; }
bool is_open(int k) { return k == MRLBM_VELOCITY || k == MRLBM_PRESSURE || k == MRLBM_VELOCITY_FD || k == MRLBM_PRESSURE_FD; }
bool is_fd(int k) { return k == MRLBM_VELOCITY_FD || k == MRLBM_PRESSURE_FD; }
bool is_velocity(int k) { return k == MRLBM_VELOCITY || k == MRLBM_VELOCITY_FD; }
// the fused kernel's face kind: FD faces take the regularized face's rho / u rule
int kernel_kind(int k) { return k == MRLBM_VELOCITY_FD ? MRLBM_VELOCITY : (k == MRLBM_PRESSURE_FD ? MRLBM_PRESSURE : k); }

} // namespace

extern "C" {

void mrlbm_default_options(mrlbm_options *o)
{
    if (!o) return;
    memset(o, 0, sizeof(*o));
    o->precision = MRLBM_FP64;
    o->device = -1;
    o->cuda_stream = nullptr;
    o->rank = 0;
    o->nranks = 1;
    o->nccl_unique_id = nullptr;
}

const char *mrlbm_status_string(mrlbm_status s)
{
    switch (s) {
    case MRLBM_OK: return "MRLBM_OK";
    case MRLBM_ERR_INVALID_ARGUMENT: return "MRLBM_ERR_INVALID_ARGUMENT";
    case MRLBM_ERR_UNSUPPORTED: return "MRLBM_ERR_UNSUPPORTED";
    case MRLBM_ERR_OUT_OF_MEMORY: return "MRLBM_ERR_OUT_OF_MEMORY";
    case MRLBM_ERR_CUDA: return "MRLBM_ERR_CUDA";
    case MRLBM_ERR_NCCL: return "MRLBM_ERR_NCCL";
    case MRLBM_ERR_NUMERICAL: return "MRLBM_ERR_NUMERICAL";
    case MRLBM_ERR_BUFFER_SIZE: return "MRLBM_ERR_BUFFER_SIZE";
    default: return "MRLBM_ERR_UNKNOWN";
    }
}

const char *mrlbm_last_error(void) { return g_last_error.c_str(); }

mrlbm_status mrlbm_nccl_unique_id(void *id128)
{
    if (!id128) return fail(MRLBM_ERR_INVALID_ARGUMENT, "id128 is NULL");
    ncclUniqueId id;
    MR_NCCL(ncclGetUniqueId(&id));
    memcpy(id128, &id, sizeof(id));
    return MRLBM_OK;
}

// Slab partition of the march axis: remainder spread over the first ranks.
// Pure host arithmetic (no CUDA), exported for the distributed tests.
mrlbm_status mrlbm_partition(int64_t n, int nranks, int rank, int64_t *n_local, int64_t *offset)
{
    if (nranks < 1 || rank < 0 || rank >= nranks || n < 1) return fail(MRLBM_ERR_INVALID_ARGUMENT, "bad partition");
    const int64_t q = n / nranks, r = n % nranks;
    *n_local = q + (rank < r ? 1 : 0);
    *offset = rank * q + std::min<int64_t>(rank, r);
    return MRLBM_OK;
}

// Validation of the create arguments without touching a GPU (exported for
// the host-logic tests).  Returns the status mrlbm_create would return.
mrlbm_status mrlbm_validate(mrlbm_lattice lattice, int64_t nx, int64_t ny, int64_t nz, double tau,
                            mrlbm_regularization reg, const mrlbm_boundary *bnd, int nranks)
{
    return mrlbm_validate_repr(lattice, nx, ny, nz, tau, reg, bnd, nranks, MRLBM_MOMENTS);
}

mrlbm_status mrlbm_validate_repr(mrlbm_lattice lattice, int64_t nx, int64_t ny, int64_t nz, double tau,
                                 mrlbm_regularization reg, const mrlbm_boundary *bnd, int nranks,
                                 mrlbm_representation repr)
{
    if (lattice < MRLBM_D2Q9 || lattice > MRLBM_D3Q27) return fail(MRLBM_ERR_INVALID_ARGUMENT, "unknown lattice");
    if (repr != MRLBM_MOMENTS && repr != MRLBM_DISTRIBUTIONS) return fail(MRLBM_ERR_INVALID_ARGUMENT, "unknown representation");
    if (reg != MRLBM_PROJECTIVE && reg != MRLBM_RECURSIVE && reg != MRLBM_BGK)
        return fail(MRLBM_ERR_INVALID_ARGUMENT, "unknown regularization");
    if (reg == MRLBM_BGK && repr == MRLBM_MOMENTS)
        return fail(MRLBM_ERR_UNSUPPORTED, "BGK is not moment-closed: use the distribution representation");
    if (repr == MRLBM_DISTRIBUTIONS && nranks != 1)
        return fail(MRLBM_ERR_UNSUPPORTED, "the distribution representation runs on one rank");
    if (!(tau > 0.5) || !std::isfinite(tau)) return fail(MRLBM_ERR_INVALID_ARGUMENT, "tau must be > 1/2 (eq 5)");
    const int D = lattice == MRLBM_D2Q9 ? 2 : 3;
    if (nx < 2 || ny < 2) return fail(MRLBM_ERR_INVALID_ARGUMENT, "nx, ny must be >= 2");
    if (D == 2 && nz != 1) return fail(MRLBM_ERR_INVALID_ARGUMENT, "D2Q9 requires nz == 1");
    if (D == 3 && nz < 2) return fail(MRLBM_ERR_INVALID_ARGUMENT, "nz must be >= 2");
    if (nx > (1 << 30) || ny > (1 << 30) || nz > (1 << 30)) return fail(MRLBM_ERR_INVALID_ARGUMENT, "extent too large");
    if (nranks < 1) return fail(MRLBM_ERR_INVALID_ARGUMENT, "nranks < 1");
    const int64_t nmarch = D == 3 ? nz : ny;
    if (nmarch / nranks < 2) return fail(MRLBM_ERR_INVALID_ARGUMENT, "each rank needs >= 2 layers along the slab axis");
    if (!bnd) return MRLBM_OK;
    for (int F = 0; F < 2 * D; F++) {
        const int k = bnd->face[F].kind;
        if (k < MRLBM_PERIODIC || k > MRLBM_PRESSURE_FD) return fail(MRLBM_ERR_INVALID_ARGUMENT, "unknown face kind");
    }
    for (int ax = 0; ax < D; ax++) {
        const bool p0 = bnd->face[2 * ax].kind == MRLBM_PERIODIC, p1 = bnd->face[2 * ax + 1].kind == MRLBM_PERIODIC;
        if (p0 != p1) return fail(MRLBM_ERR_INVALID_ARGUMENT, "periodic on only one face of an axis");
    }
    for (int F = 0; F < 2 * D; F++) {
        const mrlbm_face &f = bnd->face[F];
        if (f.kind == MRLBM_MOVING_WALL && f.u[F / 2] != 0.0)
            return fail(MRLBM_ERR_INVALID_ARGUMENT, "moving-wall velocity must be tangential");
        if (f.kind == MRLBM_MOVING_WALL && D == 2 && f.u[2] != 0.0)
            return fail(MRLBM_ERR_INVALID_ARGUMENT, "2D moving-wall velocity has a z component");
        if ((f.kind == MRLBM_PRESSURE || f.kind == MRLBM_PRESSURE_FD) && !(f.rho > 0))
            return fail(MRLBM_ERR_INVALID_ARGUMENT, "pressure face needs rho > 0");
    }
    bool any_fd = false;
    for (int F = 0; F < 2 * D; F++) any_fd |= is_fd(bnd->face[F].kind);
    if (any_fd) {
        if (repr != MRLBM_MOMENTS) return fail(MRLBM_ERR_UNSUPPORTED, "finite-difference faces need the moment representation");
        if (nranks > 1) return fail(MRLBM_ERR_UNSUPPORTED, "finite-difference faces run on one rank");
        // second-order one-sided stencils need 3 nodes along the normal and along non-periodic tangents
        const int64_t ext[3] = {nx, ny, D == 3 ? nz : 1};
        for (int ax = 0; ax < D; ax++)
            if (bnd->face[2 * ax].kind != MRLBM_PERIODIC && ext[ax] < 3)
                return fail(MRLBM_ERR_INVALID_ARGUMENT, "finite-difference faces need >= 3 nodes along bounded axes");
    }
    if (repr == MRLBM_DISTRIBUTIONS)
        for (int F = 0; F < 2 * D; F++)
            if (is_open(bnd->face[F].kind))
                return fail(MRLBM_ERR_UNSUPPORTED, "open faces are not implemented for the distribution representation");
    const int march = D == 3 ? 2 : 1;
    if (is_open(bnd->face[2 * march].kind) || is_open(bnd->face[2 * march + 1].kind))
        return fail(MRLBM_ERR_UNSUPPORTED, "open faces on the marching/slab axis are not supported");
    if (D == 3) {
        const bool ox = is_open(bnd->face[0].kind) || is_open(bnd->face[1].kind);
        const bool oy = is_open(bnd->face[2].kind) || is_open(bnd->face[3].kind);
        if (ox && oy) return fail(MRLBM_ERR_UNSUPPORTED, "open faces sharing an edge");
    }
    return MRLBM_OK;
}

mrlbm_status mrlbm_create(mrlbm_t *out, mrlbm_lattice lattice, int64_t nx, int64_t ny, int64_t nz, double tau,
                          mrlbm_regularization reg, const mrlbm_boundary *boundary, const mrlbm_options *opt)
{
    if (!out) return fail(MRLBM_ERR_INVALID_ARGUMENT, "out is NULL");
    *out = nullptr;
    mrlbm_options o;
    mrlbm_default_options(&o);
    if (opt) o = *opt;
    if (o.precision != MRLBM_FP64 && o.precision != MRLBM_FP32) return fail(MRLBM_ERR_INVALID_ARGUMENT, "precision");
    mrlbm_status st = mrlbm_validate_repr(lattice, nx, ny, nz, tau, reg, boundary, o.nranks, o.representation);
    if (st) return st;
    if (o.rank < 0 || o.rank >= o.nranks) return fail(MRLBM_ERR_INVALID_ARGUMENT, "rank out of range");

    EncodeTiledFn encode = get_encode_fn();
    if (o.device >= 0) MR_CUDA(cudaSetDevice(o.device));
    int dev = 0;
    MR_CUDA(cudaGetDevice(&dev));
    if (!encode && o.representation == MRLBM_MOMENTS) return fail(MRLBM_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");

    mrlbm_ctx *h = new mrlbm_ctx();
    h->device = dev;
    h->lattice = lattice;
    h->reg = reg;
    h->prec = o.precision;
    h->D = lattice == MRLBM_D2Q9 ? 2 : 3;
    h->M = h->D == 2 ? 6 : 10;
    h->Q = lattice == MRLBM_D2Q9 ? 9 : (lattice == MRLBM_D3Q19 ? 19 : 27);
    h->wbytes = o.precision == MRLBM_FP32 ? 4 : 8;
    h->gn[0] = nx;
    h->gn[1] = ny;
    h->gn[2] = h->D == 2 ? 1 : nz;
    h->tau = tau;
    h->omega = 1.0 - 1.0 / tau;
    h->rank = o.rank;
    h->nranks = o.nranks;
    h->repr = o.representation;
    if (boundary) h->bnd = *boundary;
    else memset(&h->bnd, 0, sizeof(h->bnd)); // all periodic

    // kernel axes: A = x, B = y (3D) / 1 (2D), C = z (3D) / y (2D)
    h->nA = (int)nx;
    h->nB = h->D == 3 ? (int)ny : 1;
    h->cglobal = (int)(h->D == 3 ? nz : ny);
    int64_t nloc, off;
    mrlbm_partition(h->cglobal, o.nranks, o.rank, &nloc, &off);
    h->nC = (int)nloc;
    h->coff = (int)off;
    // Storage: each A-row starts with padA elements (16 B) and, in 3D, each
    // moment plane with one pad row, so that every TMA box origin (tile origin
    // minus the halo) is a non-negative coordinate.  Rows are 32-B aligned.
    h->padA = 16 / h->wbytes;
    h->padB = h->D == 3 ? 1 : 0;
    const int align = 32 / h->wbytes;
    // one extra column (and, in 3D, row) after the last node: the high-side
    // periodic ghosts (the low-side ghosts live in the pads)
    h->pitch = (h->padA + h->nA + 1 + align - 1) / align * align;
    h->mstride = (long long)(h->padB + h->nB + h->padB) * h->pitch;
    h->origin = (long long)h->padB * h->pitch + h->padA;
    h->pstride = (long long)h->M * h->mstride;
    h->buf_bytes = (size_t)(h->nC + 2) * h->pstride * h->wbytes;

    auto cleanup_fail = [&](mrlbm_status s) {
        mrlbm_destroy(h);
        return s;
    };
    // the step kernels address a layer's moment planes with 32-bit offsets
    if (h->pstride >= (1LL << 31))
        return cleanup_fail(fail(MRLBM_ERR_UNSUPPORTED, "layer too large: M * (nB + 2) * pitch must stay below 2^31 elements"));

    if (o.cuda_stream) {
        h->stream = (cudaStream_t)o.cuda_stream;
    } else {
        if (cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking) != cudaSuccess)
            return cleanup_fail(fail(MRLBM_ERR_CUDA, "stream create"));
        h->own_stream = true;
    }
    if (cudaStreamCreateWithFlags(&h->cap_stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&h->ev_ready, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&h->ev_comm, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreate(&h->ev_t0) != cudaSuccess || cudaEventCreate(&h->ev_t1) != cudaSuccess)
        return cleanup_fail(fail(MRLBM_ERR_CUDA, "stream/event create"));

    if (h->repr == MRLBM_DISTRIBUTIONS) {
        // two lattices of Q shifted populations [q][z][y][x], rows 128-B aligned
        mr::StGrid &g = h->st_grid;
        g.nx = (int)nx;
        g.ny = (int)ny;
        g.nz = (int)h->gn[2];
        g.pitch = (int)((nx + 31) / 32 * 32);
        g.plane = (long long)g.ny * g.pitch;
        g.qstride = (long long)g.nz * g.plane;
        h->buf_bytes = (size_t)h->Q * g.qstride * h->wbytes;
        for (int i = 0; i < 2; i++) {
            if (cudaMalloc(&h->buf[i], h->buf_bytes) != cudaSuccess) {
                cudaGetLastError();
                return cleanup_fail(fail(MRLBM_ERR_OUT_OF_MEMORY, "state allocation failed"));
            }
            // zeros = shifted populations of the rest state f = w
            if (cudaMemsetAsync(h->buf[i], 0, h->buf_bytes, h->stream) != cudaSuccess)
                return cleanup_fail(fail(MRLBM_ERR_CUDA, "memset"));
        }
        if (cudaMalloc(&h->flag, sizeof(int)) != cudaSuccess) return cleanup_fail(fail(MRLBM_ERR_OUT_OF_MEMORY, "flag"));
        h->sv = select_st(lattice, reg, o.precision);
        mr::StArgs &a = h->st_base;
        memset(&a, 0, sizeof(a));
        a.nx = g.nx;
        a.ny = g.ny;
        a.nz = g.nz;
        a.pitch = g.pitch;
        a.plane = g.plane;
        a.qstride = g.qstride;
        a.omega = h->omega;
        a.inv_tau = 1.0 / tau;
        for (int F = 0; F < 6; F++) {
            const mrlbm_face &f = h->bnd.face[F];
            a.kind[F] = (F < 2 * h->D) ? (int)f.kind : mr::BC_PERIODIC;
            for (int q = 0; q < 3; q++) a.uw[F][q] = (F < 2 * h->D && f.kind == MRLBM_MOVING_WALL) ? f.u[q] : 0.0;
        }
        h->tilesA = (g.nx + h->sv.BX - 1) / h->sv.BX;
        h->tilesB = 1;
        h->seg_len = 1;
        h->nseg = g.ny * g.nz;
        if (cudaStreamSynchronize(h->stream) != cudaSuccess) return cleanup_fail(fail(MRLBM_ERR_CUDA, "sync"));
        *out = h;
        return MRLBM_OK;
    }

    for (int i = 0; i < 2; i++) {
        if (cudaMalloc(&h->buf[i], h->buf_bytes) != cudaSuccess) {
            cudaGetLastError();
            return cleanup_fail(fail(MRLBM_ERR_OUT_OF_MEMORY, "state allocation failed"));
        }
        if (cudaMemsetAsync(h->buf[i], 0, h->buf_bytes, h->stream) != cudaSuccess)
            return cleanup_fail(fail(MRLBM_ERR_CUDA, "memset"));
    }
    if (cudaMalloc(&h->flag, sizeof(int)) != cudaSuccess) return cleanup_fail(fail(MRLBM_ERR_OUT_OF_MEMORY, "flag"));

    // velocity profiles -> device
    for (int F = 0; F < 2 * h->D; F++) {
        mrlbm_face &f = h->bnd.face[F];
        if (is_velocity(f.kind) && f.u_profile) {
            const int ax = F / 2;
            const size_t nodes = (size_t)(nx * ny * h->gn[2]) / (size_t)h->gn[ax];
            const size_t bytes = nodes * h->D * sizeof(double);
            if (cudaMalloc(&h->prof_dev[F], bytes) != cudaSuccess) return cleanup_fail(fail(MRLBM_ERR_OUT_OF_MEMORY, "profile"));
            if (cudaMemcpy(h->prof_dev[F], f.u_profile, bytes, cudaMemcpyHostToDevice) != cudaSuccess)
                return cleanup_fail(fail(MRLBM_ERR_CUDA, "profile copy"));
        }
        f.u_profile = nullptr;
    }

    h->var = select_variant(lattice, reg, o.precision, env_int("MRLBM_TILE", 0), env_int("MRLBM_CLUSTER", 0));
    for (const void *fn : {h->var.kernel_fn, h->var.kernel_fn_push}) {
        if (!fn) continue;
        if (cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)h->var.smem) != cudaSuccess ||
            cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout,
                                 (int)cudaSharedmemCarveoutMaxShared) != cudaSuccess)
            return cleanup_fail(fail(MRLBM_ERR_CUDA, "smem attribute"));
    }
    if (o.transport == MRLBM_TRANSPORT_P2P && o.nranks > 1 && !h->var.step_push)
        return cleanup_fail(fail(MRLBM_ERR_UNSUPPORTED, "P2P transport needs the default tile (MRLBM_TILE unset)"));

    // TMA descriptors: tensor {nA, nB, M, nC + 2} of the [plane][m][b][a] layout
    for (int i = 0; i < 2; i++) {
        cuuint64_t dims[4] = {(cuuint64_t)(h->padA + h->nA + 1), (cuuint64_t)(h->padB + h->nB + h->padB),
                              (cuuint64_t)h->M, (cuuint64_t)(h->nC + 2)};
        cuuint64_t strides[3] = {(cuuint64_t)h->pitch * h->wbytes, (cuuint64_t)h->mstride * h->wbytes,
                                 (cuuint64_t)h->pstride * h->wbytes};
        cuuint32_t box[4] = {(cuuint32_t)h->var.BW, (cuuint32_t)h->var.TB, (cuuint32_t)h->M, 1};
        cuuint32_t estr[4] = {1, 1, 1, 1};
        CUresult r = encode(&h->tmap[i], h->prec == MRLBM_FP32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_FLOAT64,
                            4, h->buf[i], dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                            CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B,
                            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cleanup_fail(fail(MRLBM_ERR_CUDA, "cuTensorMapEncodeTiled failed: " + std::to_string((int)r)));
    }

    // kernel argument template: physical faces -> kernel faces A-,A+,B-,B+,C-,C+
    StepArgs &a = h->base;
    memset(&a, 0, sizeof(a));
    a.nA = h->nA;
    a.nB = h->nB;
    a.nC = h->nC;
    a.pitch = h->pitch;
    a.padA = h->padA;
    a.padB = h->padB;
    a.mstride = h->mstride;
    a.pstride = h->pstride;
    a.omega = h->omega;
    a.c_offset = h->coff;
    const int phys[6] = {0, 1, h->D == 3 ? 2 : -1, h->D == 3 ? 3 : -1, h->D == 3 ? 4 : 2, h->D == 3 ? 5 : 3};
    for (int K = 0; K < 6; K++) {
        if (phys[K] < 0) {
            a.kind[K] = mr::BC_PERIODIC;
            continue;
        }
        const mrlbm_face &f = h->bnd.face[phys[K]];
        a.kind[K] = kernel_kind(f.kind);
        if (K < 4) h->fd_face[K] = is_fd(f.kind);
        for (int q = 0; q < 3; q++) a.uw[K][q] = f.kind == MRLBM_MOVING_WALL ? f.u[q] : 0.0;
        if (K < 4) {
            a.open_drho[K] = f.rho - 1.0;
            for (int q = 0; q < 3; q++) a.open_u[K][q] = f.u[q];
            a.open_prof[K] = h->prof_dev[phys[K]];
        }
    }
    const bool perC = a.kind[4] == mr::BC_PERIODIC;
    if (h->nranks == 1) {
        a.wrapC = perC ? 1 : 0;
        a.lo_nb = a.hi_nb = perC ? 1 : 0;
    } else {
        a.wrapC = 0;
        h->nb_lo = (h->rank > 0) ? h->rank - 1 : (perC ? h->nranks - 1 : -1);
        h->nb_hi = (h->rank < h->nranks - 1) ? h->rank + 1 : (perC ? 0 : -1);
        a.lo_nb = h->nb_lo >= 0;
        a.hi_nb = h->nb_hi >= 0;
        if (a.lo_nb) a.kind[4] = mr::BC_PERIODIC; // interior cut: neighbour data in the ghost plane
        if (a.hi_nb) a.kind[5] = mr::BC_PERIODIC;
    }
    const int TA = h->var.TA, TB = h->var.TB, CL = h->var.CL;
    h->tilesA = (h->nA + TA - 3) / (TA - 2);
    // 3D: CTAs along B; a cluster of CL CTAs owns CL * TB - 2 rows
    h->tilesB = h->D == 3 ? (h->nB + CL * TB - 3) / (CL * TB - 2) * CL : 1;
    a.tilesA = h->tilesA;
    a.tilesB = h->tilesB;
    // 3D launch order: groups of MRLBM_RAST B-tiles.  Default: groups of 4 on wide
    // planes (>= 32 tiles along A, where B-neighbour tiles launched tilesA CTAs apart
    // no longer meet in L2: C5w DRAM reads 14.9 -> 13.6 GB per step, +0.3%), the
    // plain (A, B) grid otherwise (C3: groups cost 0.7-5%); profiles/r03/ab1.jsonl, ab14.jsonl
    const int rast_default = h->tilesA >= 32 ? 4 : 0;
    a.rastG = (h->D == 3 && CL == 1) ? std::max(0, env_int("MRLBM_RAST", rast_default)) : 0;
    // Segments along C.  The grid is tiles x segments; pick the segment count
    // that best fills whole waves of resident CTAs (no tail wave), preferring
    // longer segments (each segment re-reads one halo layer at each end).
    // MRLBM_SEG overrides (tuning).
    {
        const long long tiles = (long long)h->tilesA * h->tilesB;
        int occ = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, h->var.kernel_fn, h->var.TA * h->var.TB, h->var.smem);
        int nsm = 148;
        cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
        const long long slots = (long long)std::max(occ, 1) * nsm;
        long long seg = env_int("MRLBM_SEG", 0);
        if (seg <= 0 && h->D == 2) {
            // 2D: short segments keep the resident CTAs on a narrow band of
            // rows (halo rows shared by consecutive segments are L2 hits, the
            // DRAM streams stay local); each segment recomputes two halo rows.
            // Measured on C2 (profiles/segsweep_r02.jsonl, seg2d_r02.jsonl):
            // fp64 (HBM-bound) 0.84 at 24 rows -> 0.883 at 10-14; fp32
            // (issue-bound, pays the halo rows) best at 16-18.
            seg = h->prec == MRLBM_FP64 ? 12 : 16;
        } else if (seg <= 0) {
            // 3D: segment lengths 32..96; best wave fill, ties to the longer
            double best = -1.0;
            for (long long sl = std::min<long long>(96, h->nC); sl >= std::min<long long>(32, h->nC); sl--) {
                const long long ns = (h->nC + sl - 1) / sl;
                const long long units = tiles * ns;
                const long long waves = (units + slots - 1) / slots;
                const double fill = double(units) / double(waves * slots);
                const double score = fill * (double(sl) / double(sl + 2));
                if (score > best + 1e-3) {
                    best = score;
                    seg = sl;
                }
            }
        }
        seg = std::max<long long>(1, std::min<long long>(seg, h->nC));
        h->seg_len = (int)seg;
        h->nseg = (int)((h->nC + seg - 1) / seg);
    }

    h->p2p = h->nranks > 1 && o.transport == MRLBM_TRANSPORT_P2P;
    h->group_mode = h->nranks > 1 && !h->p2p && !o.nccl_unique_id;
    if (h->p2p) {
        // own sync counters (IPC-exportable cudaMalloc allocation) and error flag
        if (cudaMalloc(&h->sync, 4 * sizeof(unsigned long long)) != cudaSuccess ||
            cudaMalloc(&h->p2p_err, sizeof(int)) != cudaSuccess)
            return cleanup_fail(fail(MRLBM_ERR_OUT_OF_MEMORY, "p2p sync"));
        if (cudaMemset(h->sync, 0, 4 * sizeof(unsigned long long)) != cudaSuccess ||
            cudaMemset(h->p2p_err, 0, sizeof(int)) != cudaSuccess)
            return cleanup_fail(fail(MRLBM_ERR_CUDA, "p2p sync init"));
    }
    if (h->nranks > 1 && !h->group_mode && !h->p2p) {
        if (cudaStreamCreateWithFlags(&h->comm_stream, cudaStreamNonBlocking) != cudaSuccess)
            return cleanup_fail(fail(MRLBM_ERR_CUDA, "comm stream"));
        ncclUniqueId id;
        memcpy(&id, o.nccl_unique_id, sizeof(id));
        ncclResult_t r = ncclCommInitRank(&h->comm, h->nranks, id, h->rank);
        if (r != ncclSuccess) return cleanup_fail(fail(MRLBM_ERR_NCCL, std::string("ncclCommInitRank: ") + ncclGetErrorString(r)));
    }

    // rest state: rho = 1 (stored rho - 1 = 0), u = 0, Pi = 0 -> zeros (done by memset)
    if (cudaStreamSynchronize(h->stream) != cudaSuccess) return cleanup_fail(fail(MRLBM_ERR_CUDA, "sync"));
    *out = h;
    return MRLBM_OK;
}

void mrlbm_destroy(mrlbm_t h)
{
    if (!h) return;
    if (h->stream) cudaStreamSynchronize(h->stream);
    if (h->comm) ncclCommDestroy(h->comm);
    for (void *p : h->ipc_opened) cudaIpcCloseMemHandle(p);
    if (h->sync) cudaFree(h->sync);
    if (h->p2p_err) cudaFree(h->p2p_err);
    for (int i = 0; i < 2; i++)
        if (h->graph[i]) cudaGraphExecDestroy(h->graph[i]);
    for (int i = 0; i < 2; i++)
        if (h->buf[i]) cudaFree(h->buf[i]);
    for (int F = 0; F < 6; F++)
        if (h->prof_dev[F]) cudaFree(h->prof_dev[F]);
    if (h->io) cudaFree(h->io);
    if (h->flag) cudaFree(h->flag);
    if (h->ev_ready) cudaEventDestroy(h->ev_ready);
    if (h->ev_comm) cudaEventDestroy(h->ev_comm);
    if (h->ev_t0) cudaEventDestroy(h->ev_t0);
    if (h->ev_t1) cudaEventDestroy(h->ev_t1);
    if (h->comm_stream) cudaStreamDestroy(h->comm_stream);
    if (h->cap_stream) cudaStreamDestroy(h->cap_stream);
    if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
    delete h;
}

static int64_t local_nodes(const mrlbm_ctx *h) { return (int64_t)h->nA * h->nB * h->nC; }

mrlbm_status mrlbm_set_moments_device(mrlbm_t h, const double *src_dev, int64_t count)
{
    if (!h || !src_dev) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null argument");
    if (count != (int64_t)h->M * local_nodes(h)) return fail(MRLBM_ERR_BUFFER_SIZE, "count != M * N_local");
    if (h->p2p && !h->p2p_connected)
        return fail(MRLBM_ERR_INVALID_ARGUMENT, "P2P transport: mrlbm_p2p_connect before setting the state");
    if (h->repr == MRLBM_DISTRIBUTIONS) h->sv.set(src_dev, h->buf[h->cur], h->st_grid, h->stream);
    else h->var.set(src_dev, node0(h, h->cur), grid_args(h), h->stream);
    MR_CUDA(cudaGetLastError());
    mrlbm_status s = p2p_prologue(h);
    if (s) return s;
    MR_CUDA(cudaStreamSynchronize(h->stream)); // synchronous: src may be reused on return
    return MRLBM_OK;
}

mrlbm_status mrlbm_get_moments_device(mrlbm_t h, double *dst_dev, int64_t count)
{
    if (!h || !dst_dev) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null argument");
    if (count != (int64_t)h->M * local_nodes(h)) return fail(MRLBM_ERR_BUFFER_SIZE, "count != M * N_local");
    if (h->repr == MRLBM_DISTRIBUTIONS) h->sv.get(h->buf[h->cur], dst_dev, h->st_grid, h->stream);
    else h->var.get(node0(h, h->cur), dst_dev, grid_args(h), h->stream);
    MR_CUDA(cudaGetLastError());
    MR_CUDA(cudaStreamSynchronize(h->stream)); // synchronous: dst is complete on return
    return p2p_check(h);
}

// Host I/O of the moment representation goes through a bounded device staging
// buffer, a chunk of whole layers at a time (a 2D copy gathers the chunk's
// M strided pieces of the [M][nC][nB][nA] host array): a state that fills the
// GPU (C5 1024^3 fp64 in two copies) needs no full-size fp64 staging copy.
static const size_t kStageBytes = size_t(1) << 30;

static int64_t stage_layers(const mrlbm_ctx *h)
{
    const size_t per_layer = (size_t)h->M * h->nA * h->nB * sizeof(double);
    return std::max<int64_t>(1, std::min<int64_t>(h->nC, (int64_t)(kStageBytes / per_layer)));
}

mrlbm_status mrlbm_set_moments(mrlbm_t h, const double *src, int64_t count)
{
    if (!h || !src) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null argument");
    if (count != (int64_t)h->M * local_nodes(h)) return fail(MRLBM_ERR_BUFFER_SIZE, "count != M * N_local");
    if (h->repr == MRLBM_DISTRIBUTIONS) { // ST: one full-size staging copy
        mrlbm_status s = ensure_io(h, (size_t)count * sizeof(double));
        if (s) return s;
        MR_CUDA(cudaMemcpyAsync(h->io, src, (size_t)count * sizeof(double), cudaMemcpyHostToDevice, h->stream));
        return mrlbm_set_moments_device(h, h->io, count);
    }
    if (h->p2p && !h->p2p_connected)
        return fail(MRLBM_ERR_INVALID_ARGUMENT, "P2P transport: mrlbm_p2p_connect before setting the state");
    const int64_t plane = (int64_t)h->nA * h->nB, N = local_nodes(h), L = stage_layers(h);
    mrlbm_status s = ensure_io(h, (size_t)h->M * L * plane * sizeof(double));
    if (s) return s;
    for (int64_t c0 = 0; c0 < h->nC; c0 += L) {
        const int64_t len = std::min<int64_t>(L, h->nC - c0);
        MR_CUDA(cudaMemcpy2DAsync(h->io, (size_t)(len * plane) * sizeof(double), src + c0 * plane,
                                  (size_t)N * sizeof(double), (size_t)(len * plane) * sizeof(double), (size_t)h->M,
                                  cudaMemcpyHostToDevice, h->stream));
        mr::GridArgs g = grid_args(h);
        g.nC = (int)len;
        h->var.set(h->io, (char *)node0(h, h->cur) + (size_t)c0 * h->pstride * h->wbytes, g, h->stream);
        MR_CUDA(cudaGetLastError());
    }
    s = p2p_prologue(h);
    if (s) return s;
    MR_CUDA(cudaStreamSynchronize(h->stream));
    return MRLBM_OK;
}

mrlbm_status mrlbm_get_moments(mrlbm_t h, double *dst, int64_t count)
{
    if (!h || !dst) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null argument");
    if (count != (int64_t)h->M * local_nodes(h)) return fail(MRLBM_ERR_BUFFER_SIZE, "count != M * N_local");
    if (h->repr == MRLBM_DISTRIBUTIONS) {
        mrlbm_status s = ensure_io(h, (size_t)count * sizeof(double));
        if (s) return s;
        s = mrlbm_get_moments_device(h, h->io, count);
        if (s) return s;
        MR_CUDA(cudaMemcpyAsync(dst, h->io, (size_t)count * sizeof(double), cudaMemcpyDeviceToHost, h->stream));
        MR_CUDA(cudaStreamSynchronize(h->stream));
        return MRLBM_OK;
    }
    const int64_t plane = (int64_t)h->nA * h->nB, N = local_nodes(h), L = stage_layers(h);
    mrlbm_status s = ensure_io(h, (size_t)h->M * L * plane * sizeof(double));
    if (s) return s;
    for (int64_t c0 = 0; c0 < h->nC; c0 += L) {
        const int64_t len = std::min<int64_t>(L, h->nC - c0);
        mr::GridArgs g = grid_args(h);
        g.nC = (int)len;
        h->var.get((const char *)node0(h, h->cur) + (size_t)c0 * h->pstride * h->wbytes, h->io, g, h->stream);
        MR_CUDA(cudaGetLastError());
        MR_CUDA(cudaMemcpy2DAsync(dst + c0 * plane, (size_t)N * sizeof(double), h->io,
                                  (size_t)(len * plane) * sizeof(double), (size_t)(len * plane) * sizeof(double),
                                  (size_t)h->M, cudaMemcpyDeviceToHost, h->stream));
    }
    MR_CUDA(cudaStreamSynchronize(h->stream));
    return p2p_check(h);
}

mrlbm_status mrlbm_get_populations(mrlbm_t h, double *dst, int64_t count)
{
    if (!h || !dst) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null argument");
    if (count != (int64_t)h->Q * local_nodes(h)) return fail(MRLBM_ERR_BUFFER_SIZE, "count != Q * N_local");
    mrlbm_status s = ensure_io(h, (size_t)count * sizeof(double));
    if (s) return s;
    if (h->repr == MRLBM_DISTRIBUTIONS) h->sv.pops(h->buf[h->cur], h->io, h->st_grid, h->omega, 1.0 / h->tau, h->stream);
    else h->var.pops(node0(h, h->cur), h->io, grid_args(h), h->omega, h->stream);
    MR_CUDA(cudaGetLastError());
    MR_CUDA(cudaMemcpyAsync(dst, h->io, (size_t)count * sizeof(double), cudaMemcpyDeviceToHost, h->stream));
    MR_CUDA(cudaStreamSynchronize(h->stream));
    return MRLBM_OK;
}

mrlbm_status mrlbm_set_populations(mrlbm_t h, const double *src, int64_t count)
{
    if (!h || !src) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null argument");
    if (h->group_mode) return fail(MRLBM_ERR_UNSUPPORTED, "set_populations on a slab-group handle");
    if (h->p2p && !h->p2p_connected)
        return fail(MRLBM_ERR_INVALID_ARGUMENT, "P2P transport: mrlbm_p2p_connect before setting the state");
    const int64_t N = local_nodes(h);
    if (count != (int64_t)h->Q * N) return fail(MRLBM_ERR_BUFFER_SIZE, "count != Q * N_local");
    mrlbm_status s = ensure_io(h, (size_t)(h->Q + h->M) * N * sizeof(double));
    if (s) return s;
    MR_CUDA(cudaMemcpyAsync(h->io, src, (size_t)count * sizeof(double), cudaMemcpyHostToDevice, h->stream));
    if (h->repr == MRLBM_DISTRIBUTIONS) {
        h->sv.set_pops(h->io, h->buf[h->cur], h->st_grid, h->stream);
    } else {
        // moments of f (eqs 1-3), computed by the ST moment kernel over a dense
        // [Q][N] view of the staging buffer, then stored as the MR state
        double *mom = h->io + (size_t)h->Q * N;
        mrd::moments_of_populations(h->lattice, h->io, mom, h->nA, h->nB * h->nC, h->stream);
        MR_CUDA(cudaGetLastError());
        h->var.set(mom, node0(h, h->cur), grid_args(h), h->stream);
        mrlbm_status ps = p2p_prologue(h);
        if (ps) return ps;
    }
    MR_CUDA(cudaGetLastError());
    MR_CUDA(cudaStreamSynchronize(h->stream));
    return MRLBM_OK;
}

static const int kGraphSteps = 32; // even: a replay returns the ping-pong parity

mrlbm_status mrlbm_step(mrlbm_t h, int64_t n)
{
    if (!h || n < 0) return fail(MRLBM_ERR_INVALID_ARGUMENT, "bad step count");
    if (h->group_mode) return fail(MRLBM_ERR_INVALID_ARGUMENT, "slab-group handle: use mrlbm_step_group");
    // Batches of kGraphSteps single-rank or P2P-transport steps are replayed
    // from a captured graph (the P2P wait / signal kernels read and write the
    // device counters at run time, so a replay orders itself).  NCCL steps stay
    // eager: their launch overhead is < 1% of a C5w step, and NCCL capture
    // cannot be validated on the one-GPU test box.
    while ((h->nranks == 1 || h->p2p) && n >= kGraphSteps) {
        const int par = h->cur;
        if (!h->graph[par]) {
            cudaGraph_t g;
            MR_CUDA(cudaStreamBeginCapture(h->cap_stream, cudaStreamCaptureModeThreadLocal));
            const int64_t k0 = h->kernels;
            for (int i = 0; i < kGraphSteps; i++) {
                mrlbm_status s = enqueue_one_step(h, h->cap_stream);
                if (s) {
                    cudaStreamEndCapture(h->cap_stream, &g);
                    return s;
                }
            }
            h->graph_steps = (int)(h->kernels - k0);
            h->kernels = k0;
            MR_CUDA(cudaStreamEndCapture(h->cap_stream, &g));
            MR_CUDA(cudaGraphInstantiate(&h->graph[par], g, 0));
            cudaGraphDestroy(g);
            h->cur = par; // capture only recorded the steps
        }
        MR_CUDA(cudaGraphLaunch(h->graph[par], h->stream));
        h->kernels += h->graph_steps;
        n -= kGraphSteps;
    }
    for (int64_t i = 0; i < n; i++) {
        mrlbm_status s = enqueue_one_step(h, h->stream);
        if (s) return s;
    }
    return MRLBM_OK;
}

mrlbm_status mrlbm_sync(mrlbm_t h)
{
    if (!h) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null handle");
    MR_CUDA(cudaStreamSynchronize(h->stream));
    if (h->comm_stream) MR_CUDA(cudaStreamSynchronize(h->comm_stream));
    return p2p_check(h);
}

// ---------------------------------------------------------------- P2P transport setup
namespace {
struct P2PBlob {
    uint32_t magic;
    int32_t pid, rank, nranks, nC, prec;
    int64_t pstride, origin;
    uint64_t raw[3];                 // buf[0], buf[1], sync (same-process peers)
    cudaIpcMemHandle_t ipc[3];
};
constexpr uint32_t kP2PMagic = 0x4d525032u; // "MRP2"
static_assert(sizeof(P2PBlob) <= MRLBM_P2P_HANDLE_BYTES, "P2P handle blob too large");
} // namespace

mrlbm_status mrlbm_p2p_handle(mrlbm_t h, void *blob)
{
    if (!h || !blob) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null argument");
    if (!h->p2p) return fail(MRLBM_ERR_INVALID_ARGUMENT, "not a P2P-transport handle");
    P2PBlob b;
    memset(&b, 0, sizeof(b));
    b.magic = kP2PMagic;
    b.pid = (int32_t)getpid();
    b.rank = h->rank;
    b.nranks = h->nranks;
    b.nC = h->nC;
    b.prec = h->prec;
    b.pstride = h->pstride;
    b.origin = h->origin;
    void *ptrs[3] = {h->buf[0], h->buf[1], h->sync};
    for (int i = 0; i < 3; i++) {
        b.raw[i] = (uint64_t)(uintptr_t)ptrs[i];
        MR_CUDA(cudaIpcGetMemHandle(&b.ipc[i], ptrs[i]));
    }
    memset(blob, 0, MRLBM_P2P_HANDLE_BYTES);
    memcpy(blob, &b, sizeof(b));
    return MRLBM_OK;
}

mrlbm_status mrlbm_p2p_connect(mrlbm_t h, const void *blob_lo, const void *blob_hi)
{
    if (!h) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null handle");
    if (!h->p2p) return fail(MRLBM_ERR_INVALID_ARGUMENT, "not a P2P-transport handle");
    if ((h->nb_lo >= 0) != (blob_lo != nullptr) || (h->nb_hi >= 0) != (blob_hi != nullptr))
        return fail(MRLBM_ERR_INVALID_ARGUMENT, "neighbour handles do not match the slab's neighbours");
    MR_CUDA(cudaSetDevice(h->device));
    const size_t plane = (size_t)h->pstride * h->wbytes;
    struct Mapped { int rank; void *p[3]; };
    std::vector<Mapped> done;
    auto map = [&](const void *blob, int want_rank, Mapped &out, int &nC) -> mrlbm_status {
        P2PBlob b;
        memcpy(&b, blob, sizeof(b));
        if (b.magic != kP2PMagic || b.rank != want_rank || b.nranks != h->nranks || b.prec != h->prec ||
            b.pstride != h->pstride || b.origin != h->origin)
            return fail(MRLBM_ERR_INVALID_ARGUMENT, "P2P handle of the wrong rank or layout");
        nC = b.nC;
        for (const Mapped &m : done)
            if (m.rank == want_rank) { out = m; return MRLBM_OK; }
        out.rank = want_rank;
        for (int i = 0; i < 3; i++) {
            if (b.pid == (int32_t)getpid()) {
                out.p[i] = (void *)(uintptr_t)b.raw[i];
            } else {
                void *p = nullptr;
                cudaError_t e = cudaIpcOpenMemHandle(&p, b.ipc[i], cudaIpcMemLazyEnablePeerAccess);
                if (e != cudaSuccess) return fail(MRLBM_ERR_CUDA, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
                h->ipc_opened.push_back(p);
                out.p[i] = p;
            }
        }
        done.push_back(out);
        return MRLBM_OK;
    };
    if (blob_lo) {
        Mapped m;
        int nC = 0;
        mrlbm_status s = map(blob_lo, h->nb_lo, m, nC);
        if (s) return s;
        for (int i = 0; i < 2; i++) h->peer_plane_lo[i] = (char *)m.p[i] + plane * (size_t)(nC + 1); // its high ghost
        h->peer_sync_lo = (unsigned long long *)m.p[2];
    }
    if (blob_hi) {
        Mapped m;
        int nC = 0;
        mrlbm_status s = map(blob_hi, h->nb_hi, m, nC);
        if (s) return s;
        for (int i = 0; i < 2; i++) h->peer_plane_hi[i] = m.p[i]; // its low ghost plane 0
        h->peer_sync_hi = (unsigned long long *)m.p[2];
    }
    h->p2p_connected = true;
    return MRLBM_OK;
}


mrlbm_status mrlbm_check_finite(mrlbm_t h)
{
    if (!h) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null handle");
    MR_CUDA(cudaStreamSynchronize(h->stream));
    mrlbm_status ps = p2p_check(h);
    if (ps) return ps;
    MR_CUDA(cudaMemsetAsync(h->flag, 0, sizeof(int), h->stream));
    if (h->repr == MRLBM_DISTRIBUTIONS) h->sv.finite(h->buf[h->cur], h->st_grid, h->flag, h->stream);
    else h->var.finite(node0(h, h->cur), grid_args(h), h->flag, h->stream);
    int v = 0;
    MR_CUDA(cudaMemcpyAsync(&v, h->flag, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    MR_CUDA(cudaStreamSynchronize(h->stream));
    return v ? fail(MRLBM_ERR_NUMERICAL, "non-finite moment in the state") : MRLBM_OK;
}

mrlbm_status mrlbm_query(mrlbm_t h, int64_t *M, int64_t *Q, int64_t *n_local, int64_t *offset, int64_t *bytes)
{
    if (!h) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null handle");
    if (M) *M = h->M;
    if (Q) *Q = h->Q;
    if (n_local) *n_local = h->nC;
    if (offset) *offset = h->coff;
    if (bytes) *bytes = (int64_t)(2 * h->buf_bytes);
    return MRLBM_OK;
}

mrlbm_status mrlbm_comm_info(mrlbm_t h, int *transport, int *comm_nranks, int *comm_rank)
{
    if (!h) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null handle");
    int t = h->nranks == 1 ? 0 : (h->p2p ? 2 : (h->group_mode ? 3 : 1));
    int n = h->nranks, r = h->rank;
    if (h->comm) {
        MR_NCCL(ncclCommCount(h->comm, &n));
        MR_NCCL(ncclCommUserRank(h->comm, &r));
    }
    if (transport) *transport = t;
    if (comm_nranks) *comm_nranks = n;
    if (comm_rank) *comm_rank = r;
    return MRLBM_OK;
}

mrlbm_status mrlbm_launch_count(mrlbm_t h, int64_t *kernels)
{
    if (!h || !kernels) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null argument");
    *kernels = h->kernels;
    return MRLBM_OK;
}

mrlbm_status mrlbm_time_steps(mrlbm_t h, int64_t n, double *ms_per_step)
{
    if (!h || !ms_per_step || n < 1) return fail(MRLBM_ERR_INVALID_ARGUMENT, "bad argument");
    MR_CUDA(cudaEventRecord(h->ev_t0, h->stream));
    mrlbm_status s = mrlbm_step(h, n);
    if (s) return s;
    MR_CUDA(cudaEventRecord(h->ev_t1, h->stream));
    MR_CUDA(cudaEventSynchronize(h->ev_t1));
    float ms = 0.f;
    MR_CUDA(cudaEventElapsedTime(&ms, h->ev_t0, h->ev_t1));
    *ms_per_step = ms / (double)n;
    return MRLBM_OK;
}

// Single-process slab group: handles[r] is rank r of one decomposition created
// with nranks = n_handles and no NCCL id, all on the same device.  Per step the
// boundary planes move into the neighbours' ghost planes with device-to-device
// copies (the transport NCCL provides across GPUs), then every slab runs the
// same interior / boundary launches as the NCCL path.  All work is ordered on
// handles[0]'s stream.
mrlbm_status mrlbm_step_group(mrlbm_t *hs, int n_handles, int64_t n)
{
    if (!hs || n_handles < 2 || n < 0) return fail(MRLBM_ERR_INVALID_ARGUMENT, "bad group");
    for (int r = 0; r < n_handles; r++)
        if (!hs[r] || !hs[r]->group_mode || hs[r]->rank != r || hs[r]->nranks != n_handles ||
            hs[r]->device != hs[0]->device || hs[r]->prec != hs[0]->prec || hs[r]->pstride != hs[0]->pstride)
            return fail(MRLBM_ERR_INVALID_ARGUMENT, "handles are not ranks 0..P-1 of one slab group");
    cudaStream_t st = hs[0]->stream;
    for (int r = 1; r < n_handles; r++) {
        MR_CUDA(cudaEventRecord(hs[r]->ev_ready, hs[r]->stream));
        MR_CUDA(cudaStreamWaitEvent(st, hs[r]->ev_ready, 0));
    }
    for (int64_t t = 0; t < n; t++) {
        for (int r = 0; r < n_handles; r++) {
            mrlbm_ctx *h = hs[r];
            const size_t plane = (size_t)h->pstride * h->wbytes;
            char *mine = (char *)h->buf[h->cur];
            if (h->nb_lo >= 0) {
                mrlbm_ctx *g = hs[h->nb_lo];
                MR_CUDA(cudaMemcpyAsync(mine, (char *)g->buf[g->cur] + plane * g->nC, plane, cudaMemcpyDeviceToDevice, st));
            }
            if (h->nb_hi >= 0) {
                mrlbm_ctx *g = hs[h->nb_hi];
                MR_CUDA(cudaMemcpyAsync(mine + plane * (h->nC + 1), (char *)g->buf[g->cur] + plane * 1, plane,
                                        cudaMemcpyDeviceToDevice, st));
            }
        }
        for (int r = 0; r < n_handles; r++) {
            mrlbm_ctx *h = hs[r];
            launch_range(h, h->cur, 1, h->nC - 1, st);
            launch_boundary(h, h->cur, st, false);
        }
        for (int r = 0; r < n_handles; r++) hs[r]->cur ^= 1;
        MR_CUDA(cudaGetLastError());
    }
    MR_CUDA(cudaEventRecord(hs[0]->ev_ready, st));
    for (int r = 1; r < n_handles; r++) MR_CUDA(cudaStreamWaitEvent(hs[r]->stream, hs[0]->ev_ready, 0));
    return MRLBM_OK;
}

// Internal layout description, for the bench's roofline bookkeeping and tests:
// tile shape, segment length and grid of the fused kernel.
mrlbm_status mrlbm_kernel_config(mrlbm_t h, int *TA, int *TB, int *S, int *seg_len, int *grid_x, int *grid_y,
                                 int64_t *smem_bytes)
{
    if (!h) return fail(MRLBM_ERR_INVALID_ARGUMENT, "null handle");
    if (h->repr == MRLBM_DISTRIBUTIONS) {
        if (TA) *TA = h->sv.BX;
        if (TB) *TB = 1;
        if (S) *S = 0;
        if (seg_len) *seg_len = 1;
        if (grid_x) *grid_x = h->tilesA;
        if (grid_y) *grid_y = h->nseg;
        if (smem_bytes) *smem_bytes = 0;
        return MRLBM_OK;
    }
    if (TA) *TA = h->var.TA;
    if (TB) *TB = h->var.TB;
    if (S) *S = h->var.S;
    if (seg_len) *seg_len = h->seg_len;
    if (grid_x) *grid_x = h->tilesA * h->tilesB;
    if (grid_y) *grid_y = h->nseg;
    if (smem_bytes) *smem_bytes = (int64_t)h->var.smem;
    return MRLBM_OK;
}

} // extern "C"
