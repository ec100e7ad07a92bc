/*
 * blast_cf.h — C ABI of the B200-native BLAST corner-force library (libblastcf.so).
 *
 * The library evaluates, for Q_k-Q_{k-1} finite elements in 2D and 3D and in FP64, the generalized
 * corner force of BLAST's semi-discrete Lagrangian hydrodynamics (§2, eqs (1)-(6))
 * and returns only the right-hand sides the time integrator needs (§3.1.2: "we avoid
 * transferring the full matrix F"):
 *
 *   out_Fdot1   = F . 1           assembled into global kinematic DOFs   (momentum RHS is -F.1, eq (1);
 *                                                                         kernel 8)
 *   out_FTv     = F_z^T . v_z     per zone                               (energy RHS before M_E^{-1}, eq (2);
 *                                                                         kernel 10)
 *   out_dt_min  = min over zones and quadrature points of the time-step estimate
 *                                                     (steps 4.2 and 5; MPI min 797-798)
 *
 * with (F_z)_{ij} = sum_k alpha_k sigma(q_k) : J_z^{-1}(q_k) grad W_i(q_k) phi_j(q_k) |J_z(q_k)|  (eq (4)),
 * factored F_z = A_z B^T (eqs (5)-(6)).  The stress sigma (EOS + artificial viscosity, "see [1]",
 * PAPER.md:276-280) and the time-step formula follow the readings in DESIGN.md §3.
 *
 * Conventions (all arrays FP64 unless noted; "x fastest" lexicographic orderings):
 *   reference element [0,1]^dim; kinematic basis: tensor Lagrange on the k+1 Gauss-Lobatto-Legendre
 *   points; thermodynamic basis: tensor Bernstein of degree k-1; quadrature: tensor Gauss-Legendre with
 *   2k points per direction.  Nk = (k+1)^dim, Nt = k^dim, Nq = (2k)^dim.
 *
 * Errors: every function returns BLAST_CF_OK (0) or a positive code; blast_cf_error_string() names it
 * and blast_cf_last_error() gives a message for the most recent failure on the calling thread.
 * Asynchronous CUDA faults in an eval surface as BLAST_CF_ECUDA at the next call on the handle.
 */
#ifndef BLAST_CF_H
#define BLAST_CF_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  BLAST_CF_OK = 0,
  BLAST_CF_EINVAL = 1,       /* null / inconsistent argument */
  BLAST_CF_EUNSUPPORTED = 2, /* dim/order outside {2,3} x [1,8] */
  BLAST_CF_ENOMEM = 3,       /* device or host allocation failed */
  BLAST_CF_ECUDA = 4,        /* CUDA runtime error (launch or asynchronous fault) */
  BLAST_CF_ENCCL = 5         /* NCCL error in the multi-GPU shared-DOF exchange */
};

typedef struct blast_cf blast_cf; /* opaque; owns tables, maps, workspace and (nranks > 1) the NCCL comm */

/* The mesh as seen by ONE rank (§3.4: each MPI task owns a sub-domain).
 * All pointers are HOST pointers; the library copies what it needs at create and keeps no reference. */
typedef struct {
  int32_t dim;               /* 2 or 3 */
  int32_t order;             /* k in [1, 8]: Q_k kinematic, Q_{k-1} thermodynamic */
  int64_t num_zones;         /* zones on this rank */
  int64_t num_nodes;         /* kinematic nodes touched by this rank's zones */
  const int32_t *zone_nodes; /* [num_zones][Nk] local node ids, local node a = l0 + (k+1)(l1 + (k+1) l2) */
  const double *x0;          /* [dim][num_nodes] initial node positions (J0, h0 of the viscosity) */
  const int32_t *zone_mat;   /* [num_zones] material id, or NULL (all material 0) */
  const double *mat_gamma;   /* [num_mats] ideal-gas gamma per material */
  int32_t num_mats;
  /* domain decomposition (nranks == 1: single GPU, the fields below are ignored) */
  int32_t rank, nranks;
  int32_t num_neighbors;     /* ranks sharing at least one node with this rank */
  const int32_t *nbr_rank;   /* [num_neighbors] ascending */
  const int64_t *nbr_offset; /* [num_neighbors + 1] */
  const int32_t *nbr_nodes;  /* [nbr_offset[num_neighbors]] local node ids shared with nbr_rank[i],
                                ordered by global node id (identical order on both sides) */
} blast_cf_mesh;

/* Method constants (DESIGN.md §3 readings R8, R10, R11). */
typedef struct {
  double cfl;            /* 0.5 */
  double q_quad;         /* 2.0  quadratic viscosity coefficient */
  double q_lin;          /* 0.5  linear viscosity coefficient */
  double eps_switch;     /* 1e-12 compression-switch width */
  double h0;             /* <= 0: computed at create as (V_global / Z_global)^(1/dim) / k */
  int32_t use_viscosity; /* 1 */
  int32_t use_vorticity; /* 1: psi0 = |div v| / |grad v|_F, else 1 */
} blast_cf_params;

void blast_cf_default_params(blast_cf_params *p);

/* Create a handle.  `order` and `dim` must equal mesh->order / mesh->dim (the north-star call shape
 * blast_cf_create(mesh, order, dim)).  params NULL = defaults.  cuda_stream: a cudaStream_t (NULL =
 * the legacy default stream) on which every eval is enqueued.  nccl_unique_id: pointer to an
 * ncclUniqueId (128 bytes) shared by all ranks when mesh->nranks > 1, else NULL; the caller must have
 * selected this rank's CUDA device.  All device memory is allocated here; eval never allocates.
 * nranks > 1 with nccl_unique_id NULL creates a "loopback" handle for blast_cf_eval_loopback (tests). */
int blast_cf_create(const blast_cf_mesh *mesh, int order, int dim, const blast_cf_params *params,
                    void *cuda_stream, const void *nccl_unique_id, blast_cf **out);
/* Initial geometry (reading R19).  The viscosity length scale l = h0 |J J0^{-1} s| needs J0^{-1} at every
 * quadrature point; J varies inside a zone on curvilinear meshes (§2).  create
 * checks whether every initial zone is affine (x0 = X0 + J0 xi at all its nodes, to 1e-11 relative):
 *   affine      -> one J0^{-1} per zone ([Z][dim^2], 72 bytes/zone in 3D), the fast kernels;
 *   non-affine  -> (viscosity on) J0^{-1} at every quadrature point ([Z][Nq][dim^2], computed once on the
 *                  device from x0 by the same tensor-product basis gradients), evaluated by the generic
 *                  per-slab kernels (the only candidates that read it); h0 then uses the quadrature volume
 *                  sum_z sum_q alpha_q det J0(q). */

/* One corner-force evaluation.  All seven arrays are DEVICE pointers owned by the caller:
 *   x, v        [dim][num_nodes]  current positions and velocities (SoA)
 *   e           [num_zones][Nt]   specific internal energy, Bernstein coefficients
 *   rho0detJ0   [num_zones][Nq]   rho0(q) * det J0(q) at the quadrature points (no quadrature weight)
 *   out_Fdot1   [dim][num_nodes]  +F.1 (the momentum RHS is -F.1); on shared nodes every sharing rank
 *                                 holds the fully summed value (summed in ascending rank order)
 *   out_FTv     [num_zones][Nt]   F_z^T v_z
 *   out_dt_min  [1]               global min dt; +inf if no point has a positive inverse dt; 0 if any
 *                                 det J <= 0 (inverted zone)
 * Inputs are read-only, outputs are overwritten.  Enqueues on the handle's stream and returns without
 * synchronizing (CUDA-graph capturable for nranks == 1).  Not thread-safe per handle. */
int blast_cf_eval(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                  double *out_Fdot1, double *out_FTv, double *out_dt_min);

/* Same evaluation with HOST buffers (pinned memory recommended): copies the inputs host->device,
 * evaluates, copies the three outputs back and synchronizes the stream before returning.  Device
 * staging buffers, two internal copy streams and the zone-chunk plan are created by the first call and
 * reused.  On large meshes the copies overlap the computation chunk by chunk (zones in contiguous
 * chunks; a chunk's corner force starts when its node prefix of x, v and its e, rho0detJ0 slices have
 * arrived); the results are bitwise those of blast_cf_eval on the same data.  rho0detJ0 NULL: use the
 * copy made resident by blast_cf_set_rho0detJ0_host (no upload).  Errors: EINVAL for NULL arrays (or a
 * NULL rho0detJ0 without a resident copy), ENOMEM / ECUDA as blast_cf_eval. */
int blast_cf_eval_host(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                       double *out_Fdot1, double *out_FTv, double *out_dt_min);

/* rho0 |J0| is time-invariant (strong mass conservation, reading R2), and the paper sends only the state
 * (v, e, x) to the device each step (§3.1.2).  This copies rho0detJ0 (HOST
 * [num_zones][Nq], pinned recommended) into the handle's staging buffer once (synchronous);
 * blast_cf_eval_host(h, x, v, e, NULL, ...) then reads that resident copy instead of uploading one per
 * call.  A later call replaces it.  EINVAL for NULL. */
int blast_cf_set_rho0detJ0_host(blast_cf *h, const double *rho0detJ0);

/* Tests only: the zone-local corner force matrices F_z = A_z B^T ([num_zones][dim*Nk][Nt], device), as
 * formed by kernel 7 of the paper.  Production eval never forms them. */
int blast_cf_eval_debug_Fz(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                           double *out_Fz);

/* Tests only (single GPU): evaluate the n ranks of a domain decomposition on ONE device and run the
 * shared-DOF exchange with device copies instead of NCCL — the same pack kernel, plan (ascending-rank
 * summation) and combine kernel as the NCCL path, so partition / shared-node / ordering bugs show up
 * on one GPU.  hs[r] must have been created with mesh->rank = r, mesh->nranks = n, nccl_unique_id
 * NULL ("loopback" handle) and params->h0 > 0 (the global h0: no collective computes it).  Arrays are
 * per-rank device pointers as in blast_cf_eval.  Synchronous. */
int blast_cf_eval_loopback(blast_cf *const *hs, int n, const double *const *x, const double *const *v,
                           const double *const *e, const double *const *rho0detJ0, double *const *out_Fdot1,
                           double *const *out_FTv, double *const *out_dt_min);

/* Order-adaptive kernel selection (the paper's autotuning, §3.2.1, done at the
 * caller's request instead of over sampling periods): times every candidate corner-force kernel for the
 * handle's (dim, k) — e.g. for 3D k = 4 the warp-specialized pipeline (two register splits), the
 * CTA-synchronous DMMA kernel, the DFMA kernel and the per-slab kernel — on the given device inputs,
 * `reps` evaluations each, and keeps the fastest for all later evals.  ms_out[capacity] receives the
 * per-candidate milliseconds in candidate order, *num_candidates their count; outputs are overwritten
 * as by blast_cf_eval.  Synchronous.  blast_cf_variant_name(h, i) names candidate i (i < 0: the one
 * in use); the BLAST_CF_KB1 environment variable (a name) overrides the default at create. */
int blast_cf_autotune(blast_cf *h, const double *x, const double *v, const double *e, const double *rho0detJ0,
                      double *out_Fdot1, double *out_FTv, double *out_dt_min, int reps, double *ms_out, int capacity,
                      int *num_candidates);
const char *blast_cf_variant_name(const blast_cf *h, int index);

typedef struct {
  int32_t dim, order, nq, nk, nt;
  int64_t num_zones, num_nodes;
  double h0;                  /* the length scale in use */
  int32_t zones_per_cta, threads_per_cta, num_ctas, smem_bytes, regs_per_thread, local_bytes;
  double flops_per_zone;      /* algorithmic FP64 flops per zone: SURVEY §8(d4) F_sf */
  double alg_bytes;           /* algorithmic HBM bytes per eval */
  int32_t kernels_per_eval;   /* CUDA kernels launched by one eval */
  double flops_per_zone_alg;  /* round 1's lower flop model (6 n^3 p last stage, c_pt 420 / 160), for comparison */
} blast_cf_info;

int blast_cf_get_info(const blast_cf *h, blast_cf_info *info);

/* Per-kernel timing for the roofline report: when enabled, each eval records CUDA events around its
 * kernels on the handle's stream.  blast_cf_kernel_times() synchronizes on the last eval and returns the
 * milliseconds of [0] the corner-force kernel (KB1), [1] the node gather + dt (KB2), [2] the exchange
 * (nranks > 1, else 0) of that eval. */
int blast_cf_set_timing(blast_cf *h, int enable);
int blast_cf_kernel_times(blast_cf *h, float *ms3);

/* Multi-rank handles: which exchange schedule eval runs.
 * *mode = 0 (single rank), 1 (single round: KB1, KB2, then one grouped send/recv carrying the F.1 rows
 * and each rank's dt, so no allreduce when every rank neighbours every other) or 2 (overlap: the zones
 * touching shared nodes are numbered first — *boundary_zones of them — and run on a high-priority comm
 * stream concurrently with the interior zones, the resident CTAs split in proportion; their rows are
 * exchanged while the interior zones compute; the dt allreduce(min) overlaps the node gather).  BLAST_CF_OVERLAP=0 at create forces 1.
 * boundary_zones may be NULL. */
int blast_cf_exchange_schedule(const blast_cf *h, int32_t *mode, int64_t *boundary_zones);

/* Peer-memory transport of the exchange (SURVEY §8(e) phase 2; the MFEM shared-DOF assembly and MPI
 * min-dt of PAPER.md:772-798, the limiter named at PAPER.md:873-876).  Instead of packing the shared rows
 * for ncclSend / ncclRecv and reducing dt with ncclAllReduce, the kernel that computes a shared row stores
 * it straight into the neighbour's receive mailbox (CUDA IPC mapping: NVLink / NVSwitch loads and stores)
 * and releases a system-scope flag; each rank's dt is written into every other rank's mailbox the same
 * way; the combine kernel acquires the flags and sums in ascending rank order, so the results are bitwise
 * those of the NCCL transport.  No NCCL call is made per eval; both schedules of blast_cf_exchange_schedule
 * apply (the schedule is re-agreed at connect: overlap only if every rank can).
 * Bootstrap (collective over the caller's process group, e.g. torch.distributed with any backend):
 *   1. every rank: blast_cf_p2p_export(h, NULL, &bytes) for the record size, then
 *      blast_cf_p2p_export(h, record, &bytes) — allocates and zero-fills this rank's mailbox and describes
 *      it (IPC handle, process id, device, shared-row offsets) in `record` (host memory, `bytes` long);
 *   2. all-gather the records in rank order (rank r of the group = mesh->rank r);
 *   3. every rank: blast_cf_p2p_connect(h, records, bytes) — maps the other ranks' mailboxes
 *      (cudaIpcOpenMemHandle; plain pointers for handles of the same process) and checks that both sides
 *      of every neighbour pair agree on the shared-row counts.
 * The handle must have nranks > 1 (created with an NCCL id, or as a loopback handle: no NCCL needed at
 * all then, params->h0 must be given).  Afterwards every rank must call blast_cf_eval equally often (an
 * eval waits for its neighbours' rows of the same eval; a neighbour that never sends makes the eval's
 * kernel trap after ~30 s instead of hanging), and before blast_cf_destroy the ranks must synchronize
 * (stream sync + a process-group barrier): a peer may still be writing into this rank's mailbox until
 * its own eval has finished.  eval with a connected handle is not CUDA-graph capturable (the eval number
 * is a kernel argument).  Errors: EINVAL (bad / inconsistent records, connect twice, single-rank handle),
 * EUNSUPPORTED (no peer access between the devices), ECUDA (IPC mapping failed). */
int blast_cf_p2p_export(blast_cf *h, void *record, int64_t *bytes);
int blast_cf_p2p_connect(blast_cf *h, const void *records, int64_t bytes_each);
/* Switch a connected handle back to NCCL (enable = 0; needs the NCCL communicator of create) or to peer
 * memory again (1).  Every rank must make the same choice before its next eval — e.g. when the connect
 * failed on some rank, all ranks fall back.  Synchronizes the handle's stream.  EINVAL otherwise. */
int blast_cf_p2p_enable(blast_cf *h, int enable);
/* *transport = 0 (single rank), 1 (NCCL), 2 (loopback group, tests), 3 (peer memory, blast_cf_p2p_connect) */
int blast_cf_exchange_transport(const blast_cf *h, int32_t *transport);
/* Tests / profiling, overlap schedule with timing enabled: milliseconds from the start of the last eval to
 * [0] the end of the shared-row exchange (comm stream), [1] the end of the interior zones' corner force,
 * [2] the end of the eval.  [0] < [1] shows the exchange hidden behind the interior compute. */
int blast_cf_debug_exchange_times(blast_cf *h, float *ms3);

/* Tests only: the per-CTA minimum dt of the last eval, copied to host_out[capacity] after synchronizing
 * the stream (host_out NULL: only report the sizes).  Zone z belongs to CTA (z / zones_per_cta) mod num_ctas
 * (the corner-force kernel walks zone batches c, c + num_ctas, ... per CTA). */
int blast_cf_debug_cta_dt(blast_cf *h, double *host_out, int64_t capacity, int32_t *num_ctas, int32_t *zones_per_cta);

/* Profiling only: with BLAST_CF_PROFILE=1 in the environment at create, the corner-force kernel stamps
 * clock64() at each of its stage barriers; copies [num_ctas][16] stamps of the last eval. */
int blast_cf_debug_stage_clocks(blast_cf *h, long long *host_out, int64_t capacity);

int blast_cf_destroy(blast_cf *h);
const char *blast_cf_error_string(int code);
const char *blast_cf_last_error(void);

/* Host-only (no GPU needed), for the multi-rank tests: the exchange plan the library builds from a
 * rank's neighbour lists.  Row r of the pack buffers is the partial F.1 of nbr_nodes[r].  For every
 * shared node unique_nodes[u] (ascending local id) the partials are summed in the order
 * src[src_ptr[u] .. src_ptr[u+1]) — ascending rank — where src >= 0 is this rank's own partial (send
 * row src) and src < 0 a neighbour's (recv row -src-1).  capacity bounds unique_nodes/src_ptr/src. */
int blast_cf_exchange_plan(int32_t rank, int32_t num_neighbors, const int32_t *nbr_rank, const int64_t *nbr_offset,
                           const int32_t *nbr_nodes, int64_t capacity, int64_t *num_unique, int32_t *unique_nodes,
                           int64_t *src_ptr, int64_t *src);

/* Size of ncclUniqueId (bytes) and a helper so Python can create it without linking NCCL itself. */
/* Host-only (no CUDA): the owner weights of a rank's local nodes used by the multi-rank integrator's dot
 * products — out[n] = 0 if a neighbour with a lower rank shares node n, else 1 (each shared node is
 * counted by its lowest-ranked holder; MFEM's group masters).  Arguments as in
 * blast_cf_mesh; out: HOST [num_nodes].  EINVAL for NULL arguments or node ids out of range. */
int blast_cf_owner_mask(int32_t rank, int32_t num_neighbors, const int32_t *nbr_rank, const int64_t *nbr_offset,
                        const int32_t *nbr_nodes, int64_t num_nodes, double *out);

int blast_cf_nccl_unique_id_size(void);
int blast_cf_nccl_get_unique_id(void *out);

/* ---------------------------------------------------------------------------------------------
 * Time integrator around the corner force.
 *
 * The semi-discrete system (eqs (1)-(3))
 *     M_V dv/dt = -F.1,      M_E de/dt = F^T v,      dx/dt = v
 * with the kinematic mass matrix (M_V)_ab = int rho W_a W_b (global, sparse, solved by CG each step:
 * PAPER.md:193-198 and kernel 9 "CUDA-PCG", 405-413) and the thermodynamic mass matrix
 * (M_E)_ij = int rho phi_i phi_j (block diagonal, inverse precomputed once: PAPER.md:198-205, kernel 11,
 * 414-420).  rho|J| = rho0|J0| makes both time-independent.  Design:
 *   - M_V is never assembled: its action is evaluated matrix-free per zone by sum factorization
 *     (B^T diag(alpha rho0|J0|) B) and gathered to the nodes in ascending zone id — deterministic;
 *     Jacobi-preconditioned CG with device-resident scalars, dim systems in lockstep;
 *   - M_E^{-1}: zones whose rho0|J0| is constant over the zone use the tensor-product inverse
 *     (M1^{-1} (x) M1^{-1} (x) M1^{-1}) / (rho0|J0|) (sum-factorized); other zones a dense per-zone
 *     inverse computed at create in long double;
 *   - F^T Vbar is applied from the S(q) the corner-force kernel stores (no F_z is ever formed);
 *   - time stepping: the RK2-average scheme (reading R22), which conserves the discrete total
 *     energy 1/2 v^T M_V v + sum_z 1^T M_E e_z up to the CG tolerance (the paper's Table 6 check,
 *     PAPER.md:894-900); reflecting walls v.n = 0 on the bounding box of x0 (reading R23).
 * Multi-GPU: with a multi-rank corner-force handle every call below is collective over
 * the ranks (each process calls it for its rank; NCCL inside).  The CG for M_V adds the shared-node sum
 * of A p to every iteration (the ascending-rank exchange of blast_cf_eval) and sums its dot products over
 * the ranks with each shared node counted by its lowest-ranked holder, so all ranks keep identical
 * scalars and, on shared nodes, bitwise identical iterates; the energies are group totals.  Loopback
 * groups (n ranks on one device, tests) are driven by the *_loopback entries below.
 * --------------------------------------------------------------------------------------------- */
typedef struct blast_cf_rk2 blast_cf_rk2; /* opaque; borrows the corner-force handle h (same stream) */

typedef struct {
  double cg_rel_tol;      /* 1e-14: per component, stop when ||r|| <= tol * ||b|| (residual 2-norm) */
  int32_t cg_max_iter;    /* 500 */
  int32_t cg_check_every; /* 8: iterations between host-side convergence checks */
  int32_t wall_bc;        /* 1: v . n = 0 on the walls of the global box; 0: free */
  double box_lo[3], box_hi[3]; /* the global box of the walls; used when box_hi[0] > box_lo[0], else derived:
                                  the bounding box of x0 (one rank) or its min / max over the NCCL ranks
                                  (a collective inside create); loopback groups must give it */
} blast_cf_rk2_opts;

void blast_cf_rk2_default_opts(blast_cf_rk2_opts *o);

/* Create the integrator for handle h.  mesh: the mesh h was created from (HOST pointers; x0 gives the
 * walls).  rho0detJ0: HOST [num_zones][Nq], copied (the integrator evaluates the force with this copy).
 * Allocates all device workspace.  Multi-rank NCCL handles: collective (walls, Jacobi diagonal).
 * BLAST_CF_EUNSUPPORTED for dense M_E^{-1} zones beyond 2^34 long-double flops at create. */
int blast_cf_rk2_create(blast_cf *h, const blast_cf_mesh *mesh, const double *rho0detJ0,
                        const blast_cf_rk2_opts *opts, blast_cf_rk2 **out);

/* One RK2-average step of length dt, IN PLACE on the caller's DEVICE arrays x, v [dim][num_nodes] and
 * e [num_zones][Nt]:
 *   dv0 = -M_V^{-1} F(S0).1,  Vb = v0 + dt/2 dv0,  de0 = M_E^{-1} F(S0)^T Vb,
 *   S_half = (x0 + dt/2 Vb, Vb, e0 + dt/2 de0),
 *   dv1 = -M_V^{-1} F(S_half).1,  Vb = v0 + dt/2 dv1,  de1 = M_E^{-1} F(S_half)^T Vb,
 *   x1 = x0 + dt Vb,  v1 = v0 + dt dv1,  e1 = e0 + dt de1.
 * dt_est (HOST, may be NULL): min of the two evaluations' dt estimates (the caller's dt control);
 * cg_iters (HOST, may be NULL): CG iterations of the two solves (max over components, summed).
 * Synchronous (the CG convergence checks read device scalars). */
int blast_cf_rk2_step(blast_cf_rk2 *s, double *x, double *v, double *e, double dt, double *dt_est,
                      int32_t *cg_iters);

/* March to t_final (at most max_steps accepted steps) with the step-size control of reading R24: a step
 * whose dt estimate falls below the dt it used is undone and retried with 0.85 dt; an accepted step
 * whose estimate is >= 1.25 dt grows dt by 2 %.  *dt (HOST, in/out): the first trial dt, on return the
 * next one.  t_reached, steps, rejected (HOST, may be NULL).  x, v, e DEVICE, advanced in place. */
int blast_cf_rk2_advance(blast_cf_rk2 *s, double *x, double *v, double *e, double t_final, int32_t max_steps,
                         double *dt, double *t_reached, int32_t *steps, int32_t *rejected);

/* The two rates of the system at state (x, v, e) (DEVICE arrays): out_dvdt = -M_V^{-1} F.1 (walls
 * applied), out_dedt = M_E^{-1} F^T vbar (vbar NULL: v), out_dt = the evaluation's dt estimate (HOST).
 * Synchronous.  The building block of blast_cf_rk2_step, exposed for tests. */
int blast_cf_rk2_rates(blast_cf_rk2 *s, const double *x, const double *v, const double *e, const double *vbar,
                       double *out_dvdt, double *out_dedt, double *out_dt, int32_t *cg_iters);

/* Tests: out = M_V u per component ([dim][num_nodes], DEVICE; no wall mask). */
int blast_cf_rk2_mass_apply(blast_cf_rk2 *s, const double *u, double *out);

/* Discrete energies (HOST outputs): kinetic = 1/2 sum_c v_c^T M_V v_c, internal = sum_z 1^T M_E e_z.
 * v, e DEVICE.  Deterministic.  Synchronous. */
int blast_cf_rk2_energy(blast_cf_rk2 *s, const double *v, const double *e, double *kinetic, double *internal);

/* Tests on one device (multi-GPU logic without NCCL): S[r] is the integrator of rank r of an n-rank
 * loopback group (corner-force handles created with nranks = n and no NCCL id, opts->box_lo/box_hi set).
 * setup_loopback completes their creation (shared-node sum of the Jacobi diagonal; call once, after all
 * n creates).  rates_loopback / energy_loopback are blast_cf_rk2_rates / blast_cf_rk2_energy of the whole
 * group: per-rank DEVICE arrays, out_dt / cg_iters / kinetic / internal HOST (group values).  Synchronous. */
int blast_cf_rk2_setup_loopback(blast_cf_rk2 *const *S, int n);
int blast_cf_rk2_rates_loopback(blast_cf_rk2 *const *S, int n, const double *const *x, const double *const *v,
                                const double *const *e, const double *const *vbar, double *const *out_dvdt,
                                double *const *out_dedt, double *out_dt, int32_t *cg_iters);
int blast_cf_rk2_energy_loopback(blast_cf_rk2 *const *S, int n, const double *const *v, const double *const *e,
                                 double *kinetic, double *internal);

int blast_cf_rk2_destroy(blast_cf_rk2 *s);

#ifdef __cplusplus
}
#endif
#endif /* BLAST_CF_H */
