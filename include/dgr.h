/*
 * dgr.h — C ABI of libdgr: one RK4 stage of fp64 BSSN on a 2:1-balanced,
 * Morton-ordered octree (the data-parallel hot path of the GPU Dendro-GR
 * solver, Fernando et al., SC'22; "P:Lnnn" = line nnn of the paper text).
 *
 * The calls follow the paper's statement of the problem:
 *   Alg. 1  Require: u at t0, dt; Ensure: u at T —
 *                         halo_exchange -> octant-to-patch -> RHS ->
 *                         patch-to-octant -> AXPY            => dgr_rk4_stage / dgr_rk4_step
 *   Alg. 2  Require: octant list, O2B, u; Ensure: u^ (patches)
 *                                                             => dgr_unzip
 *   §IV-B  RHS = derivatives D + algebra A        => dgr_rhs
 *   §III-B/C octree, O2O/O2N maps, built on the host at (re)grid
 *                         time                       => dgr_octree_build, dgr_mesh_create
 *
 * Conventions
 *   - All functions are extern "C", return dgr_status, never throw.
 *   - Device pointers are plain CUDA device addresses (e.g. torch tensors'
 *     data_ptr()); `stream` is a cudaStream_t passed as void*.  Work is
 *     enqueued on `stream`; functions return before it completes unless
 *     stated otherwise.  The caller owns every state/output buffer; the
 *     library owns the mesh (host maps, device maps, workspace, NCCL
 *     communicator, streams/events) and frees it in dgr_mesh_destroy.
 *   - State layout: u[f * dof_stride + d], f = 0..23 (field order below),
 *     d = local DOF index (owned DOFs first, in global-id order, then ghost
 *     DOFs grouped by owning rank).  fp64, SoA, 16-byte aligned.
 *     Field order: 0 alpha, 1 chi, 2 K, 3-5 Gt^i, 6-8 beta^i, 9-11 B^i,
 *     12-17 gt_ij, 18-23 At_ij, ij in (xx,xy,xz,yy,yz,zz).
 *   - Patches: patches[(f * n_oct_local + e) * patch_pitch + p],
 *     p = i + 13 j + 169 k (x fastest) over the (r+2k)^3 = 13^3 padded block
 *     of P:L177 (r = 7, k = 3); patch_pitch >= 2197 (padded for alignment).
 *   - Errors: arguments are validated synchronously (DGR_ERR_ARG); bad octant
 *     lists give DGR_ERR_TREE; CUDA launch/API errors give DGR_ERR_CUDA
 *     (asynchronous faults surface at the next synchronising call).
 *     dgr_last_error() returns a thread-local message for the last failure.
 *   - A mesh handle is not thread-safe.  With nranks > 1, dgr_mesh_create,
 *     dgr_rhs, dgr_rk4_stage, dgr_rk4_step and dgr_constraints are collective:
 *     every rank calls them in the same order (NCCL semantics).
 */
#ifndef DGR_H
#define DGR_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  DGR_OK = 0,
  DGR_ERR_ARG = -1,    /* null/misaligned pointer, bad size or index          */
  DGR_ERR_TREE = -2,   /* octants unsorted, overlapping, incomplete, unbalanced */
  DGR_ERR_CUDA = -3,   /* CUDA runtime error                                   */
  DGR_ERR_NCCL = -4,   /* NCCL unavailable or failed                          */
  DGR_ERR_OOM = -5,    /* host or device allocation failed                    */
  DGR_ERR_STATE = -6   /* call not valid for this mesh (e.g. host-only mesh)  */
} dgr_status;

/* Leaf octant: anchor in units of width / 2^max_depth, level l has side
 * 2^(max_depth - l) in those units (leaves only). 16 bytes. */
typedef struct {
  uint32_t x, y, z;
  uint32_t level;
} dgr_octant;

/* Puncture for the refinement rule (DESIGN.md R-O1). */
typedef struct {
  double x, y, z, m;
  int32_t level; /* finest level required at the puncture */
  int32_t pad;
} dgr_puncture;

/* Inputs of dgr_octree_build: refine every octant while
 *   level < max(level_min, max_a [L_a - j_a]),  j_a = min j>=0 with
 *   d^2(box, x_a) <= (rho m_a)^2 4^j,
 * then apply the minimal 2:1 vertex-balance closure and sort by Morton key
 * (child index c = x + 2y + 4z). */
typedef struct {
  double xmin[3];
  double width;
  int32_t max_depth; /* <= 20; 18 in all shipped configs */
  int32_t periodic;  /* 1: periodic domain, 0: extrapolating outer boundary */
  int32_t level_min;
  int32_t n_punct;
  const dgr_puncture* punct; /* host array [n_punct] */
  double rho;
} dgr_refine_desc;

/* Mesh creation options. */
typedef struct {
  double xmin[3];
  double width;
  int32_t max_depth;
  int32_t periodic;
  int32_t rank, nranks;   /* Morton-contiguous partition of the leaves     */
  int32_t device;         /* 1: upload maps + allocate workspace on the current
                             CUDA device; 0: host-only (maps/export only)  */
  int32_t pad;
  const void* nccl_id;    /* ncclUniqueId bytes (128) when nranks > 1; NULL with
                             nranks > 1 selects external-exchange mode: no
                             communicator, the caller refreshes the ghost DOFs
                             itself (DGR_MAP_SEND / _COUNTS) before each stage */
} dgr_mesh_desc;

/* Parameters of the RHS (readings R6, R8, R13, R29). */
typedef struct {
  double ko_sigma;   /* Kreiss-Oliger strength sigma (0.4)                  */
  double eta;        /* Gamma-driver damping eta (2.0), eq (3)              */
  double lambda_f0;  /* f(alpha) = lambda_f0 + lambda_f1 alpha, eq (2) (1,0) */
  double lambda_f1;
  double chi_floor;  /* chi in every division is max(chi, chi_floor) (1e-4) */
  int32_t sommerfeld; /* 1: radiative outer boundary at the DOFs on the faces of a
                         non-periodic domain, d_t f = -(x^i/r) d_i f - (f - f_inf)/r
                         (reading R29; PAPER.md is silent); 0: none (default) */
  int32_t upwind;     /* 1: advective derivatives beta^k d_k f by the 4th-order lopsided
                         stencil (-3 f_-1 - 10 f_0 + 18 f_1 - 6 f_2 + f_3)/(12 h) shifted
                         towards +k where beta^k >= 0, mirrored where < 0 (reading R9u,
                         for long moving-puncture evolutions); 0: centred D1 (R9,
                         default; the paper's 72 first derivatives) */
} dgr_params;

typedef struct {
  int64_t n_oct_global;
  int64_t n_oct_local;   /* owned octants of this rank                      */
  int64_t n_oct_ghost;   /* ghost octants (remote padding/hanging sources)   */
  int64_t oct_begin;     /* global index of the first owned octant           */
  int64_t n_dof_global;
  int64_t n_dof_owned;
  int64_t n_dof_ghost;
  int64_t dof_stride;    /* >= n_dof_owned + n_dof_ghost, multiple of 32     */
  int64_t patch_pitch;   /* doubles per patch (>= 2197)                      */
  int64_t n_hanging;     /* hanging (octant, node) pairs over local+ghost    */
  double h_min;          /* finest grid spacing width / (6 * 2^level_max)    */
  int32_t level_min, level_max;
  int64_t n_interp_slots;  /* interpolation slots (hanging nodes + coarse-neighbour
                              padding values, deduplicated; device meshes only) */
  int64_t n_interp_elems;  /* elements whose slots k_interp evaluates          */
  int64_t n_oct_interior;  /* owned octants whose patches need no ghost value
                              (computed while the ghost exchange is in flight,
                              SURVEY.md §8e; = n_oct_local on one rank)        */
} dgr_mesh_info;

typedef struct dgr_mesh_s* dgr_mesh;

/* Canonical map exports (host buffers, global indices; bit-exact contract
 * with the oracle). */
enum {
  DGR_MAP_OCTANTS = 0,  /* int32 [n_oct_global][4]: x, y, z, level (Morton order)  */
  DGR_MAP_O2N = 1,      /* int32 [n_oct_local][343]: global DOF id or -1 (hanging)  */
  DGR_MAP_HANGING = 2,  /* int32 [n][3]: (global octant, node, global source leaf)
                           over owned octants, sorted by (octant, node)            */
  DGR_MAP_PAD_SRC = 3,  /* int32 [n_oct_local][2197]: global source leaf, -1 = extrap */
  DGR_MAP_PAD_KIND = 4, /* uint8 [n_oct_local][2197]: 0 self, 1 copy, 2 inject,
                           3 interp, 4 extrap; | 8 if reached across the periodic
                           boundary                                                */
  DGR_MAP_ZIP = 5,      /* int32 [n_dof_owned][2]: (global owner leaf, node)       */
  DGR_MAP_DOF_GID = 6,  /* int64 [n_dof_owned + n_dof_ghost]: global DOF id        */
  DGR_MAP_DOF_XYZ = 7,  /* double [3][n_dof_owned + n_dof_ghost]: coordinates      */
  DGR_MAP_SEND = 8,     /* int32 [sum over peers]: local DOF ids sent, peer-major   */
  DGR_MAP_SEND_COUNTS = 9, /* int64 [nranks]: DOFs sent to each peer               */
  DGR_MAP_RECV_COUNTS = 10, /* int64 [nranks]: ghost DOFs received from each peer  */
  DGR_MAP_LOCAL_OCTS = 11,  /* int32 [n_oct_local + n_oct_ghost]: global octant ids */
  DGR_MAP_O2N_LOCAL = 12,   /* int32 [n_oct_local + n_oct_ghost][343]: local DOF id or -1 */
  DGR_MAP_RHS_ORDER = 13,   /* int32 [n_oct_local]: owned octants (local ids) in RHS order,
                               the first n_oct_interior need no ghost value (device meshes) */
  DGR_MAP_SENDBUF = 14      /* double [sum_p NF * n_p]: the send buffer of the last ghost
                               exchange, peer-major — for peer p a [NF][n_p] block, row f
                               holding u[f][DGR_MAP_SEND entries of p] (test hook; device
                               meshes; synchronises the device) */
};

const char* dgr_status_string(dgr_status s);
const char* dgr_last_error(void);
const char* dgr_version(void);

/* Host: refine + balance + Morton sort.  Call with out = NULL to get
 * the count in *n_inout; then with a buffer of *n_inout entries. */
dgr_status dgr_octree_build(const dgr_refine_desc* desc, dgr_octant* out, int64_t* n_inout);

/* Host (+device when desc->device): validate the octant list (sorted,
 * complete, non-overlapping, 2:1 vertex balanced -> else DGR_ERR_TREE), build
 * node/DOF numbering, hanging table, padding (O2P) and zip maps, partition
 * along the Morton curve for `rank` of `nranks`, upload maps, allocate
 * workspace.  Synchronises `stream`. */
dgr_status dgr_mesh_create(const dgr_mesh_desc* desc, const dgr_octant* octs, int64_t n,
                           void* stream, dgr_mesh* out);
dgr_status dgr_mesh_info_get(dgr_mesh m, dgr_mesh_info* info);
/* Copy map `which` to host_buf; with host_buf = NULL return the size in *nbytes. */
dgr_status dgr_mesh_export_maps(dgr_mesh m, int which, void* host_buf, size_t* nbytes);
dgr_status dgr_mesh_destroy(dgr_mesh m);

/* Device: coordinates of the local DOFs, xyz[a * dof_stride + d]. */
dgr_status dgr_dof_coords(dgr_mesh m, double* xyz, void* stream);

/* Device: octant-to-patch (Alg. 2) of the first `nfields` fields of u into
 * patches (layout above).  Single-rank meshes, or u whose ghost DOFs are
 * current (see dgr_ghost_exchange). */
dgr_status dgr_unzip(dgr_mesh m, const double* u, double* patches, int nfields, void* stream);

/* Device: ghost exchange of all 24 fields of u (Alg. 1 line 5 halo_exchange,
 * P:L215; NCCL, nranks > 1; no-op with one rank).  The owned DOFs each peer
 * needs are packed into a peer-major send buffer (one [24][n_p] block per peer
 * p, DGR_MAP_SEND order), exchanged as ONE grouped ncclSend/ncclRecv pair per
 * peer, and unpacked into u's ghost slice (DOFs n_dof_owned.., grouped by
 * owning rank).  DGR_ERR_STATE on meshes without a communicator
 * (external-exchange mode: the caller refreshes the ghosts; grouped meshes:
 * dgr_group_ghost_exchange); NCCL failures give DGR_ERR_NCCL. */
dgr_status dgr_ghost_exchange(dgr_mesh m, double* u, void* stream);

/* Device: BSSN RHS (eqs 1-8 + KO) at the interior points of given patches
 * (24 fields, layout above) -> rhs_oct[(f * n_oct_local + e) * 343 + n]. */
dgr_status dgr_rhs_patches(dgr_mesh m, const double* patches, double* rhs_oct,
                           const dgr_params* prm, void* stream);

/* Device: F(u) on the owned DOFs: ghost exchange -> unzip -> RHS -> zip.
 * rhs[f * dof_stride + d] for owned d.  u must be writable when nranks > 1
 * (its ghost slice is refreshed). */
dgr_status dgr_rhs(dgr_mesh m, double* u, double* rhs, const dgr_params* prm, void* stream);

/* Device: RK4 stage s = 0..3 (classic tableau, reading R11).  Reads the
 * stage state U_s (= u_n for s = 0; pass u_s == u_n), computes k = F(U_s) and
 *   s=0: acc = u_n + dt/6 k; u_s = u_n + dt/2 k      s=1: acc += dt/3 k; u_s = u_n + dt/2 k
 *   s=2: acc += dt/3 k;      u_s = u_n + dt k        s=3: acc += dt/6 k   (acc = u^{n+1})
 * All three arrays are [24][dof_stride].  For s = 0, u_s may alias u_n only
 * if the caller does not need u_n's ghost DOFs afterwards. */
dgr_status dgr_rk4_stage(dgr_mesh m, int s, double dt, double* u_n, double* u_s, double* acc,
                         const dgr_params* prm, void* stream);

/* Device: one RK4 step in place on u (library workspace for stages).
 * nranks > 1 needs a communicator: on an external-exchange or grouped mesh it
 * returns DGR_ERR_STATE (step those with dgr_rk4_stage + the caller's ghost
 * refresh, or dgr_group_rk4_step).  dgr_rhs, dgr_rk4_stage and dgr_constraints
 * do work on external-exchange meshes: they read the ghost DOFs as given. */
dgr_status dgr_rk4_step(dgr_mesh m, double dt, double* u, const dgr_params* prm, void* stream);

/* Host buffers: one RK4 step (as dgr_rk4_step) of each of n independent
 * host-resident states on this mesh, u_out[j] = step(u_in[j]), j = 0..n-1
 * (Alg. 1 with the state on the host, for callers without device
 * memory; u_in[j] == u_out[j] is allowed).  Each u_in[j] / u_out[j] is a host
 * array in the device state layout, [24][dof_stride] doubles; rows are read
 * and written for the owned DOFs d < n_dof_owned only (ghost values come from
 * the exchange).  Page-locked (cudaHostAlloc / torch pin_memory) buffers are
 * required for the copies to overlap: the host->device copy of state j+1 and
 * the device->host copy of state j-1 run on two library copy streams while
 * state j steps on `stream`, through three library-owned device state slots
 * (allocated on first use, 3 x 24 x dof_stride doubles).  Enqueued on `stream`
 * like the device calls: u_out[j] is complete when `stream` is; the host
 * arrays must stay valid until then.  n == 0 is a no-op; a null list or entry
 * is DGR_ERR_ARG.  Collective when nranks > 1 (every rank passes the same n). */
dgr_status dgr_rk4_step_host(dgr_mesh m, double dt, int64_t n, const double* const* u_in,
                             double* const* u_out, const dgr_params* prm, void* stream);

/* Device: constraints H, M^0..2, G^0..2 on the owned DOFs,
 * c[q * dof_stride + d], q = 0..6; norms_host[2q] = RMS, [2q+1] = max |.|
 * over owned DOFs (all ranks).  Synchronises `stream`. */
dgr_status dgr_constraints(dgr_mesh m, double* u, double* c, double* norms_host,
                           const dgr_params* prm, void* stream);

/* The paper's code-generation study (§IV-B, Table II; SURVEY
 * §8(f) row 3) — not the default path (dgr_rhs fuses the derivatives with the
 * algebra and never stores them):
 * dgr_rhs_inputs: the 234 inputs of the algebraic part A at every interior
 *   point of the owned octants, in[k * ld + e * 343 + p] (ld >= n_oct_local *
 *   343): k < 24 field values, then 72 first derivatives (24 + 3 f + a), 66
 *   second derivatives of alpha, chi, beta^i, gt_ij (96 + 6 s + q, q over
 *   xx xy xz yy yz zz), 72 Kreiss-Oliger terms (162 + 3 f + a, scaled by
 *   sigma / (64 h)) — the layout of codegen/bssn_sym.py.  Ghost exchange +
 *   unzip into the library's patch buffer + one derivative kernel.
 * dgr_rhs_algebra: out[f * ld + i] = A_f + KO_f at n points of in (same ld) by
 *   the generated kernel `variant`: 0 SymPyGR-style global CSE, 1 binary
 *   reduction over the expression DAG (Alg. 3), 2 staged CSE; occ = 1 selects
 *   the occupancy-constrained build (256 threads x 4 CTAs, <= 64 registers,
 *   the analogue of the paper's __launch_bounds__(343,3)).  Device pointers;
 *   no mesh. */
dgr_status dgr_rhs_inputs(dgr_mesh m, double* u, double* in, int64_t ld, const dgr_params* prm,
                          void* stream);
dgr_status dgr_rhs_algebra(int variant, int occ, const double* in, double* out, int64_t n,
                           int64_t ld, const dgr_params* prm, void* stream);

/* Regrid (Alg. 1 line 3 construct_grid; refinement tolerance
 * P:L465; the paper delegates it to DENDRO-GR without formulas: readings
 * R30-R32 of DESIGN.md).
 * dgr_regrid_indicator: w[e] (device, n_oct_local doubles) = the wavelet
 *   indicator of owned octant e — the largest |P - prediction| over the interior
 *   points of its 13^3 patches of the fields in field_mask (bit f = field f),
 *   the prediction being the tensor degree-6 Lagrange interpolant from the
 *   all-even patch points (spacing 2h).  0 up to rounding for data of degree
 *   <= 6 per axis.  Ghost exchange + unzip + one kernel.
 * dgr_regrid_octree: host; the regridded leaves from w (host, n_oct_global
 *   doubles, global Morton order): a leaf with w > eps_refine and level <
 *   level_max is split, a complete family of 8 sibling leaves with every w <
 *   eps_coarsen and level > level_min (none split) is merged, then the minimal
 *   2:1 vertex-balance closure and Morton order (every leaf changes by at most
 *   one level).  out = NULL returns the count in *n_inout (as dgr_octree_build).
 * dgr_regrid_transfer: u_new (the new mesh's state, owned DOFs) = the old
 *   mesh's piecewise interpolant at every new DOF: the tensor Lagrange
 *   interpolant of the finest old leaf containing it (lowest Morton on ties),
 *   hanging nodes reconstructed; copies where a new DOF is an old node.  Both
 *   meshes single-rank, same domain; synchronises `stream`. */
dgr_status dgr_regrid_indicator(dgr_mesh m, double* u, uint32_t field_mask, double* w,
                                void* stream);
dgr_status dgr_regrid_octree(dgr_mesh m, const double* w, double eps_refine, double eps_coarsen,
                             int level_min, int level_max, dgr_octant* out, int64_t* n_inout);
dgr_status dgr_regrid_transfer(dgr_mesh old_m, double* u_old, dgr_mesh new_m, double* u_new,
                               void* stream);

/* Gravitational-wave extraction ("the Penrose scalar Psi_4 ... expanded
 * in spin-weighted spherical harmonics (l, m modes) on spherical shells";
 * readings R33-R36 of DESIGN.md).
 * dgr_psi4: psi[c * ld + e * 343 + node] (device, ld = n_oct_local * 343, c = 0
 *   Re, 1 Im) = Psi_4 = (E_ij - i B_ij) mbar^i mbar^j at every node of every
 *   owned octant, from that octant's own patch (E, B the electric / magnetic
 *   Weyl parts in vacuum; tetrad r^, theta^, phi^ about center[3],
 *   Gram-Schmidt in the physical metric).  Ghost exchange + unzip + the
 *   234-input derivative kernel + the generated k_psi4.
 * dgr_psi4_sphere: host points xyz[3][npts] (physical) -> out[2][npts] (host):
 *   the degree-6 interpolant of psi over the finest octant containing each
 *   point (single-rank meshes; synchronises).
 * dgr_psi4_modes: the whole extraction on a sphere of `radius` about center:
 *   Gauss-Legendre (n_theta) x uniform (n_phi) quadrature (reading R35, in
 *   place of Lebedev's), modes[2 q], [2 q + 1] = Re, Im of C_lm = sum_k w_k
 *   Psi_4(x_k) conj(-2Y_lm(x_k)), q over l = 2..l_max, m = -l..l; `sphere`
 *   (host [2][n_theta * n_phi], optional) receives the point values. */
dgr_status dgr_psi4(dgr_mesh m, double* u, const double* center, double* psi,
                    const dgr_params* prm, void* stream);
dgr_status dgr_psi4_sphere(dgr_mesh m, const double* psi, int64_t npts, const double* xyz,
                           double* out, void* stream);
dgr_status dgr_psi4_modes(dgr_mesh m, double* u, const double* center, double radius, int n_theta,
                          int n_phi, int l_max, double* modes, double* sphere,
                          const dgr_params* prm, void* stream);

/* In-process rank group: n meshes of one octree, meshes[r] = rank r of n,
 * each created with nccl_id = NULL (one per device, or several on one device),
 * driven by ONE process.  Their ghost exchange is libdgr's own (SURVEY §8e
 * with the NCCL transport replaced): the same peer-major pack kernel and send
 * buffers as dgr_ghost_exchange, one cudaMemcpyPeerAsync per (rank, peer)
 * pair into the peer's receive buffer (NVLink between devices), the same
 * unpack kernel.  The group borrows the meshes: destroy it before them
 * (dgr_mesh_destroy of a grouped mesh is DGR_ERR_STATE).  u[r] / streams[r]:
 * rank r's state and cudaStream_t (arrays of n); streams may coincide. */
typedef struct dgr_group_s* dgr_group;
dgr_status dgr_group_create(dgr_mesh* meshes, int n, dgr_group* out);
/* ghost exchange of every rank's u[r]; complete on streams[r] */
dgr_status dgr_group_ghost_exchange(dgr_group g, double* const* u, void* const* streams);
/* one RK4 step in place on every u[r] (as dgr_rk4_step), the exchange of each
 * stage overlapped with the interior octants of every rank */
dgr_status dgr_group_rk4_step(dgr_group g, double dt, double* const* u, const dgr_params* prm,
                              void* const* streams);
dgr_status dgr_group_destroy(dgr_group g);

/* Execution options of a mesh (host-side switch, takes effect at the next call):
 *   DGR_OPT_FUSED_UNZIP (default 1): 1 = dgr_rhs / dgr_rk4_* gather every patch
 *     inside the RHS kernel straight from the element values and interpolation
 *     slots (no patch buffer); 0 = unzip into the 13^3 patch
 *     buffer first (Alg. 2), then the RHS reads the patches.
 *     Both give bit-identical results. */
/*   DGR_OPT_PHASES (default 0): how the fused path orders the owned octants.
 *     0 = interior octants overlap the ghost exchange when there is a
 *     communicator, else one pass; 1 = always run the interior octants (and the
 *     slots they need) first, then the rest; 2 = interior octants only (test
 *     hook: boundary octants' RHS is not computed). */
/*   DGR_OPT_PREPASS (default 1): fused path without the radiative boundary
 *     evaluates the six gt_ij fields' derivatives in a separate metric pre-pass
 *     kernel (two CTAs per SM, 30 values per point through HBM) and the other
 *     18 fields in the RHS kernel; 0 = all 24 fields in the RHS kernel.  Both
 *     give bit-identical results. */
/*   DGR_OPT_ZIP_STORE (default 1): fused path without the radiative boundary
 *     zips in the RHS kernel's store (each point writes its 24 values to the
 *     DOF it is the zip owner of) and the RK4 update streams the
 *     DOF-ordered RHS; 0 = RHS per octant point, then the zip gather (k_zip /
 *     k_zip_rk4).  Both give bit-identical results. */
/*   DGR_OPT_GRAPH (default 1): dgr_rk4_step replays a CUDA graph of its four
 *     stages: the first call with given (u, dt, params) runs eagerly, the second
 *     captures the launch sequence on a library stream, later calls launch the
 *     graph on `stream` (one launch instead of 16+).  Changing any option or
 *     the arguments re-captures.  Not used while profiling (dgr_profile_enable)
 *     or on NCCL meshes.  Bit-identical to the eager sequence. */
/*   DGR_OPT_FUSE_RK4 (default 1): dgr_rk4_step and dgr_rk4_step_host apply the
 *     RK4 stage update (Alg. 1 l.9-10, classic tableau) in the RHS kernel's
 *     zip-by-store epilogue — each zip owner updates its DOF's stage state and
 *     accumulator (or the new state) instead of storing the RHS, the u_n /
 *     accumulator rows prefetched into L2 two field stages ahead — with stage
 *     states alternating between two library buffers; 0 = the RHS in DOF order,
 *     then a streaming update kernel.  Fused path with zip by store only;
 *     dgr_rk4_stage and the rank group always use the separate update.
 *     Bit-identical. */
enum { DGR_OPT_FUSED_UNZIP = 1, DGR_OPT_PHASES = 2, DGR_OPT_PREPASS = 3, DGR_OPT_ZIP_STORE = 4,
       DGR_OPT_GRAPH = 5, DGR_OPT_FUSE_RK4 = 7 };
dgr_status dgr_set_option(dgr_mesh m, int option, int64_t value);

/* Device-side timing helper for benchmarks: number of kernel launches the last
 * dgr_rk4_step / dgr_rhs enqueued. */
int64_t dgr_last_launch_count(dgr_mesh m);

/* Per-kernel device timing: when enabled, every libdgr launch is bracketed by
 * CUDA events recorded on the launching stream.  dgr_profile_read synchronises
 * and returns, per kernel class, the summed milliseconds and launch counts
 * since the last reset (classes: 0 elements, 1 hanging, 2 unzip, 3 rhs,
 * 4 zip/zip+rk4, 5 ghost pack/exchange, 6 constraints, 7 interp (coarse-neighbour
 * padding values of the fused unzip)). */
enum { DGR_PROF_CLASSES = 8 };
dgr_status dgr_profile_enable(dgr_mesh m, int on);
dgr_status dgr_profile_read(dgr_mesh m, double* ms, int64_t* counts, int reset);

/* fp64 FMA throughput microbenchmark on the current device: `blocks` CTAs of
 * 256 threads, each thread running 8 independent DFMA chains for `iters`
 * iterations.  Returns the elapsed device milliseconds and the FLOP count
 * (2 per DFMA).  Used to measure the fp64 roofline denominator. */
dgr_status dgr_bench_dfma(int blocks, int iters, void* stream, double* ms, double* flops);

#ifdef __cplusplus
}
#endif
#endif /* DGR_H */
