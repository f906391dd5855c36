/*
 * mrlbm.h -- C ABI of the B200-native moment-representation regularized
 * lattice Boltzmann library (libmrlbm.so).
 *
 * The method: Valero-Lara, Vetter, Gounley, Randles, "Moment Representation
 * of Regularized Lattice Boltzmann Methods on NVIDIA and AMD GPUs" (SC'23 W).
 * Citations "P:Lnnn" are lines of that paper's text; "Rk" are the
 * readings of ambiguous passages listed in DESIGN.md.
 *
 * State (Alg. 2 lines 7-8, 16-23): per lattice
 * node the M = 1 + D + D(D+1)/2 moments
 *     2D (M=6):  rho, u_x, u_y, Pi_xx, Pi_yy, Pi_xy
 *     3D (M=10): rho, u_x, u_y, u_z, Pi_xx, Pi_yy, Pi_zz, Pi_xy, Pi_xz, Pi_yz
 * rho = sum f (eq 1), u = (sum c f)/rho (eq 2; velocity, R5), Pi the Hermite
 * second moment sum (c c - c_s^2 I) f (eq 3, c_s^2 = 1/3).  These are the
 * post-streaming (= pre-collision) moments.  One mrlbm_step = collide
 * (regularized, eqs 8-14) + stream (eq 7) + boundary treatment, computed by
 * one fused sm_100a kernel that reads and writes only these moments.
 *
 * Host array layout (all host I/O is fp64, C order, caller-owned):
 *     moments      [M][nz_local][ny][nx]   (2D: [M][ny][nx])
 *     populations  [Q][nz_local][ny][nx]   (2D: [Q][ny][nx])
 * Velocity ordering (paper silent; R1): index 0 = rest, then a positive half,
 * then its negation (opp(i) = i +- (Q-1)/2):
 *   D2Q9 : (1,0) (0,1) (1,1) (1,-1)
 *   D3Q19: (1,0,0) (0,1,0) (0,0,1) (1,1,0) (1,-1,0) (1,0,1) (1,0,-1) (0,1,1) (0,1,-1)
 *   D3Q27: the D3Q19 half, then (1,1,1) (1,1,-1) (1,-1,1) (1,-1,-1)
 *
 * Errors: every function returns an mrlbm_status (0 = OK, < 0 = error) and
 * leaves a thread-local message for mrlbm_last_error().  No function aborts
 * the process.  Handles are not thread-safe; several handles may coexist.
 */
#ifndef MRLBM_H
#define MRLBM_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct mrlbm_ctx *mrlbm_t; /* opaque; owns all device memory it allocates */

typedef enum { MRLBM_D2Q9 = 0, MRLBM_D3Q19 = 1, MRLBM_D3Q27 = 2 } mrlbm_lattice;

/* projective: eqs 8-11; recursive: eqs 8, 10, 12-14
 * with Malaspinas' recursion [8] (R8) and the per-lattice basis R10.
 * BGK: the single-relaxation-time collision of the paper's standard reference
 * (Alg. 1 lines 21-25, eq 4 per R2); it is not moment-closed, so it
 * exists only with MRLBM_DISTRIBUTIONS (MRLBM_ERR_UNSUPPORTED with MOMENTS). */
typedef enum { MRLBM_PROJECTIVE = 0, MRLBM_RECURSIVE = 1, MRLBM_BGK = 2 } mrlbm_regularization;

/* State representation.
 *   MOMENTS       (default) the paper's method (MR, Alg. 2): M moments per node,
 *                 2 M w bytes per lattice update (Table 2).
 *   DISTRIBUTIONS the paper's comparison baseline (ST, Alg. 1): Q
 *                 pre-collision populations per node in two lattices, 2 Q w
 *                 bytes per update; one push kernel per step (collide + stream,
 *                 walls as the MR path).  Single rank; periodic / wall /
 *                 moving-wall faces only (open faces: MRLBM_ERR_UNSUPPORTED).
 * Both expose the same state through the same calls (moments = eqs 1-3 of the
 * pre-collision populations) and give the same trajectory for the regularized
 * collisions up to rounding. */
typedef enum { MRLBM_MOMENTS = 0, MRLBM_DISTRIBUTIONS = 1 } mrlbm_representation;

/* Arithmetic and storage precision of the device state.  FP64 is the paper's
 * (P:L257); FP32 stores rho - 1 and shifted populations (R16). */
typedef enum { MRLBM_FP64 = 0, MRLBM_FP32 = 1 } mrlbm_precision;

/* Halo transport between z-slab ranks (nranks > 1):
 *   NCCL  per step, ncclSend/ncclRecv of one boundary plane per face on a
 *         communication stream, overlapped with the interior layers.
 *   P2P   the fused step itself stores its first / last layer straight into
 *         the neighbours' ghost planes through peer memory (CUDA IPC; NVLink
 *         between GPUs), and device-side counters in peer memory order the
 *         steps (no NCCL call, no separate copy).  Ranks may share a device
 *         (then the peer "link" is local memory).  Requires
 *         mrlbm_p2p_handle / mrlbm_p2p_connect before the first step. */
typedef enum { MRLBM_TRANSPORT_NCCL = 0, MRLBM_TRANSPORT_P2P = 1 } mrlbm_transport;

/* Face treatment ("bounceback ... at the channel walls", inlet/outlet
 * per Latt et al. [6]; readings R12-R14):
 *   PERIODIC     both faces of an axis must be periodic
 *   WALL         halfway link-wise bounce-back, wall at -1/2 and n-1/2
 *   MOVING_WALL  WALL plus the Ladd momentum term 2 w_i rho (c_i.u_w)/c_s^2,
 *                rho = the node's pre-collision density; u_w tangential
 *   VELOCITY     regularized velocity face: u prescribed (u[] or u_profile)
 *   PRESSURE     regularized pressure face: rho prescribed, tangential u = 0
 *   VELOCITY_FD, PRESSURE_FD
 *                finite-difference faces of Latt et al. [6], the inlet /
 *                outlet of the paper's proxy apps ("finite difference
 *                boundary conditions at the inlet and outlet"; R20): rho and u
 *                as above, Pi^neq = -rho tau c_s^2 (grad u + grad u^T) of the
 *                new velocity field by second-order differences (one-sided
 *                along the normal and at the face's edges, central elsewhere).
 *                One rank, MOMENTS only (else MRLBM_ERR_UNSUPPORTED); >= 3
 *                nodes along every non-periodic axis (else INVALID_ARGUMENT).
 *                Runs as a separate face kernel after the fused step.
 * Open faces (VELOCITY/PRESSURE[_FD]) are supported on the x and y faces of 3D
 * domains and on the x faces of 2D domains (not on the marching / slab axis). */
typedef enum {
    MRLBM_PERIODIC = 0, MRLBM_WALL = 1, MRLBM_MOVING_WALL = 2,
    MRLBM_VELOCITY = 3, MRLBM_PRESSURE = 4,
    MRLBM_VELOCITY_FD = 5, MRLBM_PRESSURE_FD = 6
} mrlbm_bc_kind;

typedef struct {
    mrlbm_bc_kind kind;
    double u[3];             /* MOVING_WALL / VELOCITY (uniform) velocity */
    double rho;              /* PRESSURE density */
    const double *u_profile; /* optional, VELOCITY[_FD] only: [face nodes][D], host,
                                row-major over the two other axes (slower axis
                                first; global, not slab-local); copied at create */
} mrlbm_face;

typedef struct {
    mrlbm_face face[6]; /* order: x-, x+, y-, y+, z-, z+ (z ignored in 2D) */
} mrlbm_boundary;

typedef struct {
    mrlbm_precision precision; /* default FP64 */
    int device;                /* CUDA device ordinal, default current (-1) */
    void *cuda_stream;         /* cudaStream_t to enqueue on; NULL = own stream */
    int rank, nranks;          /* z-slab decomposition (2D: y-slabs); default 0, 1 */
    const void *nccl_unique_id;/* 128-byte ncclUniqueId for nranks > 1 (one GPU per
                                  rank); NULL with nranks > 1 = slab-group mode */
    mrlbm_representation representation; /* default MOMENTS */
    mrlbm_transport transport;  /* nranks > 1: halo transport, default NCCL (see below) */
} mrlbm_options;

typedef int mrlbm_status;
#define MRLBM_OK 0
#define MRLBM_ERR_INVALID_ARGUMENT -1 /* tau <= 1/2, n < 2, D2Q9 with nz != 1, one-sided periodic, bad kind */
#define MRLBM_ERR_UNSUPPORTED -2      /* open faces sharing an edge, open face on the marching axis;
                                         BGK with MOMENTS; DISTRIBUTIONS with open faces or nranks > 1;
                                         a layer of M * (ny + 2) * pitch >= 2^31 elements (3D in-plane
                                         sizes beyond ~14000^2: the step kernels use 32-bit offsets) */
#define MRLBM_ERR_OUT_OF_MEMORY -3
#define MRLBM_ERR_CUDA -4
#define MRLBM_ERR_NCCL -5
#define MRLBM_ERR_NUMERICAL -6        /* non-finite moment found by mrlbm_check_finite */
#define MRLBM_ERR_BUFFER_SIZE -7      /* count != M * N_local (or Q * N_local) */

/* Fill mrlbm_options with defaults (FP64, current device, own stream, 1 rank). */
void mrlbm_default_options(mrlbm_options *opt);

/* Create a solver for an nx x ny (x nz) box with relaxation time tau (eq 5).
 * The state is initialised to rest (rho = 1, u = 0, Pi = 0).  With
 * nranks > 1 the dimensions are GLOBAL and the library owns the contiguous
 * z-slab (2D: y-slab) of this rank; neighbours exchange one boundary plane
 * of moments per step through NCCL send/recv.
 * boundary may be NULL (fully periodic); opt may be NULL (defaults). */
mrlbm_status mrlbm_create(mrlbm_t *out, mrlbm_lattice lattice, int64_t nx, int64_t ny, int64_t nz,
                          double tau, mrlbm_regularization reg, const mrlbm_boundary *boundary,
                          const mrlbm_options *opt);

/* Copy a host moment field (layout above, this rank's slab) into the device
 * state.  count must equal M * N_local.  Synchronous. */
mrlbm_status mrlbm_set_moments(mrlbm_t h, const double *src, int64_t count);

/* Advance n timesteps (n >= 0).  Asynchronous: enqueues on the handle's stream
 * (batches of steps are replayed from a captured CUDA graph). */
mrlbm_status mrlbm_step(mrlbm_t h, int64_t n);

/* Copy the current moments to host (layout above).  Synchronises the stream. */
mrlbm_status mrlbm_get_moments(mrlbm_t h, double *dst, int64_t count);

/* Post-collision populations f* of the current state (eqs 9 / 14; R17),
 * [Q][nz_local][ny][nx] fp64 on host.  count must equal Q * N_local. */
mrlbm_status mrlbm_get_populations(mrlbm_t h, double *dst, int64_t count);

/* Set the state from PRE-collision populations f, [Q][nz_local][ny][nx] fp64
 * host, count = Q * N_local.  DISTRIBUTIONS stores them as they are.  MOMENTS
 * stores their moments (eqs 1-3): the regularized collisions read only those
 * (P:L49), so the trajectory is the same.  Synchronous. */
mrlbm_status mrlbm_set_populations(mrlbm_t h, const double *src, int64_t count);

/* Device-side variants for zero-copy I/O: dst/src are DEVICE pointers to fp64
 * arrays in the host layout above.  The copy runs on the handle's stream and
 * the call returns after it completed (synchronous, like the host variants):
 * the caller must have finished writing src (e.g. synchronised the stream that
 * produced it) and may reuse or free the buffer as soon as the call returns.
 * On a P2P-transport handle the set variants require mrlbm_p2p_connect first
 * (MRLBM_ERR_INVALID_ARGUMENT otherwise: the neighbours' ghost planes could
 * not be filled). */
mrlbm_status mrlbm_set_moments_device(mrlbm_t h, const double *src_dev, int64_t count);
mrlbm_status mrlbm_get_moments_device(mrlbm_t h, double *dst_dev, int64_t count);

/* Wait for all enqueued work.  P2P transport: MRLBM_ERR_CUDA if a halo wait
 * timed out (a neighbour stopped); the handle then refuses further steps. */
mrlbm_status mrlbm_sync(mrlbm_t h);

/* Halo transport of a handle: *transport = 0 single rank, 1 NCCL, 2 P2P,
 * 3 slab group; for NCCL *comm_nranks / *comm_rank are what the communicator
 * reports (ncclCommCount / ncclCommUserRank), else nranks / rank. */
mrlbm_status mrlbm_comm_info(mrlbm_t h, int *transport, int *comm_nranks, int *comm_rank);

/* Scan the state for non-finite values (debug aid); MRLBM_ERR_NUMERICAL if any
 * (MRLBM_ERR_CUDA first if a P2P halo wait timed out). */
mrlbm_status mrlbm_check_finite(mrlbm_t h);

/* Sizes: M, Q, local march extent, its global offset, device bytes held. */
mrlbm_status mrlbm_query(mrlbm_t h, int64_t *M, int64_t *Q, int64_t *n_local, int64_t *offset,
                         int64_t *bytes);

/* Launch statistics since creation: kernels enqueued by mrlbm_step and the
 * number of CUDA graph replays (for the bench's gpu_launches count). */
mrlbm_status mrlbm_launch_count(mrlbm_t h, int64_t *kernels);

/* Time one step's fused kernel launches with CUDA events on the handle's
 * stream (device milliseconds per step, averaged over n steps). */
mrlbm_status mrlbm_time_steps(mrlbm_t h, int64_t n, double *ms_per_step);

void mrlbm_destroy(mrlbm_t h);
const char *mrlbm_status_string(mrlbm_status s);
const char *mrlbm_last_error(void); /* thread-local detail of the last error */

/* Write a 128-byte ncclUniqueId into id (rank 0 creates it, then it is
 * broadcast out of band, e.g. through torch.distributed). */
mrlbm_status mrlbm_nccl_unique_id(void *id128);

/* P2P transport setup (options.transport = MRLBM_TRANSPORT_P2P, nranks > 1).
 * mrlbm_p2p_handle writes this rank's MRLBM_P2P_HANDLE_BYTES-byte handle
 * (CUDA IPC handles of its two state buffers and its sync counters, plus raw
 * pointers used when the neighbour lives in the same process) into blob;
 * distribute them out of band (e.g. torch.distributed all_gather).
 * mrlbm_p2p_connect maps the handles of the lower / upper z neighbour (NULL
 * where the slab has none: non-periodic ends); both may be the same rank.
 * Collective: every rank connects before any rank steps.  Errors:
 * MRLBM_ERR_INVALID_ARGUMENT (not a P2P handle, wrong neighbour rank or
 * layout), MRLBM_ERR_CUDA (IPC mapping failed).  A neighbour that stops
 * stepping makes this rank's next step give up after 30 s; mrlbm_sync then
 * returns MRLBM_ERR_CUDA. */
#define MRLBM_P2P_HANDLE_BYTES 512
mrlbm_status mrlbm_p2p_handle(mrlbm_t h, void *blob);
mrlbm_status mrlbm_p2p_connect(mrlbm_t h, const void *blob_lo, const void *blob_hi);

/* Slab-group mode (one process, one device): handles created with nranks = P,
 * rank = r and nccl_unique_id = NULL form one z-slab decomposition whose halo
 * planes are exchanged with device-to-device copies instead of NCCL.  Advance
 * all P slabs by n steps (enqueued on handles[0]'s stream; each handle's own
 * stream is ordered before and after).  mrlbm_step on such a handle returns
 * MRLBM_ERR_INVALID_ARGUMENT.  Used to verify the decomposition on one GPU. */
mrlbm_status mrlbm_step_group(mrlbm_t *handles, int n_handles, int64_t n);

/* Host-only helpers (no CUDA calls): the slab partition of an extent n over
 * nranks (remainder to the first ranks), and the argument validation that
 * mrlbm_create performs (returns the status mrlbm_create would return). */
mrlbm_status mrlbm_partition(int64_t n, int nranks, int rank, int64_t *n_local, int64_t *offset);
mrlbm_status mrlbm_validate(mrlbm_lattice lattice, int64_t nx, int64_t ny, int64_t nz, double tau,
                            mrlbm_regularization reg, const mrlbm_boundary *boundary, int nranks);
/* The same for a given representation (mrlbm_validate = MOMENTS). */
mrlbm_status mrlbm_validate_repr(mrlbm_lattice lattice, int64_t nx, int64_t ny, int64_t nz, double tau,
                                 mrlbm_regularization reg, const mrlbm_boundary *boundary, int nranks,
                                 mrlbm_representation representation);

/* Fused-kernel launch configuration of a handle (tile TA x TB threads, TMA
 * stages S, sweep segment length, grid, dynamic shared memory bytes).  For
 * DISTRIBUTIONS: TA = threads per block along x, TB = 1, S = 0, seg_len = 1,
 * grid_x = blocks along x, grid_y = ny * nz, smem 0. */
mrlbm_status mrlbm_kernel_config(mrlbm_t h, int *TA, int *TB, int *S, int *seg_len, int *grid_x, int *grid_y,
                                 int64_t *smem_bytes);

#ifdef __cplusplus
}
#endif
#endif /* MRLBM_H */
