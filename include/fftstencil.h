/*
 * fftstencil.h -- C ABI of the B200-native FlashFFTStencil hot path.
 *
 * The library computes `total_steps` time steps of a d-dimensional (d = 1, 2, 3)
 * FP64 stencil with fixed boundary cells, by the FFT route of FlashFFTStencil
 * (PAPER.md /root/reference/PAPER.md):
 *   - the grid is split into overlap-save tiles, halo h = radius*T  (§3.1 Splitting,
 *     Eq. 3, Eq. 4; Stitching Eq. 7);
 *   - each pair of real tiles is packed as one complex tile (Double-layer Filling,
 *     §3.2.3 Eq. 9), transformed axis by axis (Algorithm 1) with
 *     each length-L DFT reshaped into small DFTs (§3.2.1: Cooley-Tukey per
 *     axis; 1D prime-factor map Eq. 8 L214-L218 for short grids) that run either as
 *     butterflies on the FP64 ALU (default: on B200 the FP64 tensor path equals and
 *     shares the DFMA budget, reading Q20) or as DFT GEMMs on the FP64
 *     tensor cores (DMMA; FFTSTENCIL_ENGINE=dmma), multiplied by the stencil spectrum raised to the power T
 *     (temporal fusion §4 Eq. 10), inverse-transformed, cropped and stored,
 *     all inside one fused kernel (Kernel Tailoring, §3.1 Fusing L190-L198);
 *   - cells within h of the fixed ring are recomputed by T direct steps (the paper is
 *     silent on boundaries; reading Q5).
 * The result equals the plain definition (PAPER.md: each step, a cell becomes the
 * weighted sum of its neighbours) up to FP64 rounding.
 *
 * Conventions (all entry points):
 *   ndim       1, 2 or 3.
 *   extents    ndim int64 values, outermost axis first; the grid is C-order contiguous
 *              FP64 and INCLUDES the fixed ring; every extent must exceed 2*radius.
 *   weights    (2*radius+1)^ndim FP64 values in offset-cube row-major order (axis 0
 *              outermost): weights[((o0+r)*(2r+1) + (o1+r))*(2r+1) + (o2+r)] multiplies
 *              u[c+o] (correlation form, reading Q1).  Star stencils are boxes
 *              with zeros.  Copied at plan creation; the caller keeps ownership.
 *   radius     1..8.
 *   T          requested fused depth (time steps per FFT pass), >= 1; 0 = automatic.
 *              The plan may lower T to fit its tile; the chosen value is in plan_info.
 *   ring       cells with some coordinate c_a < radius or c_a >= extents[a]-radius keep
 *              their input value at every step (reading Q2).
 * Errors: functions returning int give FFTSTENCIL_OK (0) or a negative code;
 * functions returning a pointer give NULL.  Either way fftstencil_last_error() then
 * describes the failure (thread-local, never NULL, "" when the last call succeeded).
 * Asynchronous device faults surface at the caller's next synchronisation.
 */
#ifndef FFTSTENCIL_H
#define FFTSTENCIL_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum {
  FFTSTENCIL_OK = 0,
  FFTSTENCIL_EINVAL = -1,        /* invalid argument                               */
  FFTSTENCIL_ENOMEM = -2,        /* host or device allocation failed               */
  FFTSTENCIL_ECUDA = -3,         /* a CUDA runtime call or kernel launch failed    */
  FFTSTENCIL_ENCCL = -4,         /* an NCCL call of the multi-GPU halo exchange failed */
  FFTSTENCIL_EUNSUPPORTED = -5   /* valid request this build does not implement    */
};

/* Opaque plan: owns its device auxiliary data (DFT matrices, powered spectra, band
 * blocks) and one grid-sized device scratch buffer.  Bound to the CUDA device that
 * was current at creation.  Not re-entrant: one fftstencil_run at a time per plan. */
typedef struct fftstencil_plan fftstencil_plan;

typedef struct {
  int ndim;
  int T;                        /* fused steps per pass actually used               */
  int radius;
  int halo;                     /* h = radius*T                                     */
  int tile[3];                  /* FFT tile extent per axis (1D: N1*N2 in tile[0])  */
  int valid[3];                 /* S = tile - 2h, cells each tile stores per axis   */
  int pfa[2];                   /* 1D prime-factor split N1 x N2 (0 otherwise)      */
  int64_t extents[3];
  int64_t tiles;                /* overlap-save tiles covering the exact region     */
  int64_t pairs;                /* complex tile pairs (Double-layer Filling)        */
  int64_t band_blocks;          /* CTA blocks of the boundary-band kernel           */
  double flops_per_cell_step;   /* algorithmic FP64 flops per cell-step (the plan's
                                   dense-DFT tile, unpadded)  */
  double mma_flops_per_pass;    /* FP64 tensor flops one fused-kernel launch issues
                                   (padding included)                               */
  size_t smem_bytes;            /* dynamic shared memory of the fused kernel        */
  size_t device_bytes;          /* device memory the plan owns                      */
  int fused_grid;               /* CTAs of the persistent fused kernel              */
  int64_t last_run_launches;    /* kernels the last fftstencil_run enqueued          */
  /* outer-axis decomposition (single GPU: nranks = 1, the whole grid) */
  int nranks, rank;
  int64_t row_begin, row_end;   /* global axis-0 rows this rank owns (its in/out slab)  */
  int64_t pair_begin, pair_end; /* tile pairs this rank computes                         */
  int64_t interior_begin, interior_end; /* pairs needing no halo rows (overlap the exchange) */
  int64_t ghost_lo, ghost_hi;   /* halo rows received from rank-1 / rank+1 per pass     */
  int algo;                     /* tile algorithm: 0 dense L^d DFT GEMMs, 1 factored (2D 64 =
                                   8 x 8, 3D 16 = 8 x 2 Cooley-Tukey), 2 unfused 2D ablation
                                   (FFTSTENCIL_ALGO=unfused: forward / multiply / inverse as
                                   three kernels with the spectrum in HBM)                  */
  int periodic;                 /* 1 for a FFTSTENCIL_PERIODIC plan                      */
  int engine;                   /* line-DFT engine of the factored tile (algo 1): 0 DFT GEMMs
                                   on the FP64 tensor pipe (DMMA), 1 butterflies in registers
                                   on the FP64 ALU (default; FFTSTENCIL_ENGINE=dmma|alu)      */
  double alu_ops_per_pass;      /* engine 1: FP64 ALU instructions one fused launch executes
                                   (adds, multiplies and FMAs, each one)                    */
  int last_run_pipelined;       /* 1 if the last fftstencil_run_host overlapped its copies with
                                   row-skewed passes (pipelined schedule), 0 if it ran plain
                                   copy-run-copy (FFTSTENCIL_E2E_PIPE=0, 1D, small grids, h > S) */
  int last_run_chunks;          /* that run's pipelined schedule: K input / output row chunks   */
  int last_run_depth;           /*   and Q skewed passes at each end (0 / 0 when not pipelined) */
  int last_run_peer_fused;      /* peer transport: 1 if the last run's boundary rows reached the
                                   neighbours as the kernels' own stores, 0 (copy pushes / other)  */
} fftstencil_info;

/* Plan creation flags (fftstencil_plan_create_ex / fftstencil_describe_ex). */
enum {
  FFTSTENCIL_PERIODIC = 1   /* periodic boundary instead of the fixed ring: every cell is updated,
                               neighbours wrap modulo the extents; single GPU */
};

/* Build a plan (host precompute + device upload).  Returns NULL on error.
 * What it computes: the tile size and fused depth T (the role of Eq. 5, re-derived
 * as a B200 cost model), the per-axis DFT tables (Algorithm 1 inputs F, L254),
 * the powered spectra S_t = sigma^t / prod(L) for t = 1..T (Eq. 10; reading Q6/Q7), the
 * overlap-save tile schedule (Eq. 3, Eq. 4) and the boundary band blocks; only the
 * tile-sized auxiliary data is kept on the device (L200: 2(2L^2+L), not the grid's).
 * Ownership: the caller keeps `extents` and `weights`; the plan owns its device memory.
 * Errors: NULL + last_error (EINVAL for bad arguments, ECUDA / ENOMEM on device failure). */
fftstencil_plan* fftstencil_plan_create(int ndim, const int64_t* extents, const double* weights,
                                        int radius, int T);

/* As fftstencil_plan_create with creation `flags` (FFTSTENCIL_PERIODIC or 0). */
fftstencil_plan* fftstencil_plan_create_ex(int ndim, const int64_t* extents, const double* weights,
                                           int radius, int T, int flags);

/* The hot path.  Enqueue `total_steps` (>= 0) time steps on `stream` (a cudaStream_t; NULL =
 * the legacy default stream): floor(total_steps / T) fused passes with S_T and one with
 * S_(total_steps mod T) (the temporal driver, §4, Fig. 2 left L111-L128; reading
 * Q15), each pass = per tile pair: halo'd load, forward DFT, * S_t, inverse DFT, crop and
 * stitch (Algorithm 1, Stitching Eq. 7) in one kernel (Fusing L190-L198),
 * plus the band cells' direct steps (reading Q5).  `in` and `out` are device pointers to prod(extents) FP64
 * values on the plan's device; the caller owns them.  `in` is read only unless it
 * aliases `out` (allowed).  total_steps == 0 copies in to out.  Asynchronous: no host
 * synchronisation.  Returns FFTSTENCIL_OK or a negative code.
 * Launches: per fused pass the tile kernel (+ the band kernel on a side stream, joined
 * before the next pass); a small non-periodic 1D grid (PFA tile, <= 8192 cells) runs the
 * whole call as ONE launch of an 8-CTA cluster with the grid in shared memory
 * (kernel_small1d.cu; FFTSTENCIL_SMALL1D=0 disables). */
int fftstencil_run(fftstencil_plan* plan, const double* in, double* out, int64_t total_steps,
                   void* stream);

/* Flexible outputs (§4: results at chosen time steps): outs[k] receives
 * the state after emit_steps[k] steps (non-decreasing, >= 0), k = 0..n_emit-1; each segment
 * is fused independently (remainder pass per segment).  Device buffers; outs must not alias
 * each other; `in` may alias outs[0].  Asynchronous on `stream`. */
int fftstencil_run_emit(fftstencil_plan* plan, const double* in, const int64_t* emit_steps, int n_emit,
                        double* const* outs, void* stream);

/* End-to-end variant with HOST buffers: copies h_in (prod(extents) FP64, pageable or
 * pinned) to device, runs, copies the result to h_out, and synchronises `stream`
 * before returning.  Uses two device grids owned by the plan (allocated on first use).
 * Single-GPU 2D/3D fixed-boundary plans with >= 2K outer tile rows overlap the copies with
 * the passes (DESIGN.md §6 "pipelined run_host"): the input arrives in K outer-row chunks
 * while the first Q passes advance row-skewed behind it, and the last Q passes finish the
 * result chunk by chunk while earlier chunks are copied out; results are bitwise equal to
 * fftstencil_run.  The copies run on a plan-owned stream ordered after / before `stream`.
 * Environment: FFTSTENCIL_E2E_PIPE=K (default 6..12 by grid size, 0 = plain copy-run-copy),
 * FFTSTENCIL_E2E_DEPTH=Q (default 16 for 2D, 20 for 3D plans), FFTSTENCIL_E2E_DEPTH_TAIL (tail
 * depth, default Q), FFTSTENCIL_E2E_RAMP (1), FFTSTENCIL_E2E_BAND_SMS (SMs left to the band, 4);
 * fftstencil_plan_info reports the K / Q the last call took. */
int fftstencil_run_host(fftstencil_plan* plan, const double* h_in, double* h_out,
                        int64_t total_steps, void* stream);

/* ---- multi-GPU: outer-axis (axis 0) domain decomposition, one process per GPU ----
 * The grid is cut into nranks slabs of whole overlap-save tile rows (2D/3D) or tile pairs
 * (1D), so every rank computes exactly the single-GPU tiles and results are bitwise
 * identical to fftstencil_run on one GPU.  `extents` are GLOBAL; `in`/`out` passed to
 * fftstencil_run are this rank's slab: rows [row_begin, row_end) of fftstencil_plan_info
 * (every slab must hold at least radius*T rows).  Before every fused pass each rank swaps
 * h = radius*T halo rows with rank-1 and rank+1 by NCCL send/recv on a library-owned
 * stream over NVLink; tile pairs whose inputs need no halo run concurrently with the
 * exchange.  `nccl_unique_id` is the 128-byte ncclUniqueId of the group (rank 0 creates it
 * with fftstencil_nccl_unique_id and broadcasts it); creation is collective over the
 * ranks.  nranks = 1 gives an ordinary plan.  nccl_unique_id = NULL creates a LOOPBACK
 * rank: no communicator; the ranks of one process are then run together on one device by
 * fftstencil_run_group, which exchanges halos by device copies (tests the decomposition
 * without several GPUs).  Returns NULL on error (ENCCL failures included). */
fftstencil_plan* fftstencil_plan_create_dist(int ndim, const int64_t* extents, const double* weights,
                                             int radius, int T, int nranks, int rank,
                                             const void* nccl_unique_id);

/* ---- peer-memory transport: the same decomposition without NCCL ----
 * Each rank's two slab buffers and a two-word flag array are shared with its neighbours through
 * CUDA IPC.  In every pass the kernels that produce a rank's h = radius*T boundary rows (the edge
 * tile pairs and the band) store those cells straight into the neighbours' halo rows as well
 * (NVLink stores; same-device stores when processes share one GPU) -- or, for the DMMA engines
 * and FFTSTENCIL_PEER_FUSED=0, the rows are copied there after the pass -- and the rank then
 * bumps the neighbours' flag word with a stream memory write; before its
 * halo-dependent tile pairs a rank's stream waits (stream memory wait, no host round trip, no
 * spinning kernel) until both neighbours have signalled as often as it has.  Halo-free pairs
 * run before the wait, so the exchange overlaps them.  Results are bitwise equal to one GPU.
 * Every rank must make the same sequence of fftstencil_run calls (same total_steps): the
 * ranks advance in lockstep (P + 1 signals per run of P passes).
 * Creation is local (no collective); then each rank exports its handle
 * (fftstencil_peer_handle, FFTSTENCIL_PEER_HANDLE_BYTES), the ranks exchange them (any host
 * channel: torch.distributed, files, ...) and each connects to its neighbours
 * (fftstencil_peer_connect: lower = rank-1's handle or NULL for rank 0, upper = rank+1's or NULL
 * for the last rank).  fftstencil_run before connecting fails with EINVAL.  The devices of
 * neighbouring ranks must be peer capable (NVLink/NVSwitch), or the same device; connect probes
 * a peer copy and a stream-memory write and fails (ECUDA) if either does not work, so the caller
 * can still choose another transport.  Errors: a run that fails midway leaves the ranks out of
 * lockstep -- destroy the group's plans.  Destroy: every rank's stream work must be finished
 * (e.g. synchronise, then a host barrier) before any rank destroys its plan, because the
 * neighbours write into its buffers. */
#define FFTSTENCIL_PEER_HANDLE_BYTES 256
fftstencil_plan* fftstencil_plan_create_dist_peer(int ndim, const int64_t* extents, const double* weights,
                                                  int radius, int T, int nranks, int rank);
int fftstencil_peer_handle(const fftstencil_plan* plan, void* out, int64_t cap);
int fftstencil_peer_connect(fftstencil_plan* plan, const void* lower, const void* upper);

/* Host-only: the op list a peer-transport run of rank `rank` executes (capi.cu run_dist_peer; the
 * op codes are in csrc/plan.h build_peer_schedule: WAIT / COPYIN / PUSH / SIGNAL / INTERIOR /
 * EDGE / COPYOUT), for `total_steps` steps, fused stores or copy pushes, after `epoch0` earlier
 * signals; 4 int64 per op.  `out` holds `cap` ops (NULL queries the count).  Returns the number
 * of ops or a negative code.  For CPU replays of the multi-rank protocol (tests/test_dist.py). */
int64_t fftstencil_peer_schedule(int ndim, const int64_t* extents, const double* weights, int radius,
                                 int T, int nranks, int rank, int64_t total_steps, int fused,
                                 int64_t epoch0, int64_t* out, int64_t cap);

/* Writes a new 128-byte ncclUniqueId into `out` (caller-owned, >= 128 bytes; rank 0 of a
 * group).  ENCCL if NCCL cannot create one.  No PAPER.md passage: the paper is single-GPU;
 * the decomposition is SURVEY §8(a) row a10. */
int fftstencil_nccl_unique_id(void* out);

/* Runs loopback ranks 0..nranks-1 (plans[k] created with rank k, nccl_unique_id NULL, on the
 * current device) for total_steps, in[k]/out[k] being rank k's device slabs; enqueued on
 * `stream`.  Asynchronous like fftstencil_run. */
int fftstencil_run_group(fftstencil_plan* const* plans, const double* const* in, double* const* out,
                         int nranks, int64_t total_steps, void* stream);

/* Host-only: the slab geometry rank `rank` of `nranks` would get (see fftstencil_info). */
int fftstencil_describe_dist(int ndim, const int64_t* extents, const double* weights, int radius,
                             int T, int nranks, int rank, fftstencil_info* info);

/* Release everything the plan owns (device tables, scratch grids, streams, events, the NCCL
 * communicator).  NULL is a no-op.  Must not race a pending fftstencil_run on the plan:
 * synchronise its stream first. */
void fftstencil_destroy(fftstencil_plan* plan);

/* Plan geometry and cost model (tile, valid window S = L - 2h of Eq. 4 / reading Q4, T,
 * pair counts of Eq. 9, algorithmic flops per cell-step, FP64 ALU instructions per launch,
 * launches of the last run).  `info` is caller-owned.  EINVAL for NULL arguments. */
int fftstencil_plan_info(const fftstencil_plan* plan, fftstencil_info* info);

/* Per-kernel timing for roofline reporting.  With profiling enabled, fftstencil_run
 * records a CUDA event pair on its stream around every fused FFT-tile launch and every
 * band launch (event overhead only; no synchronisation).  fftstencil_profile_read waits
 * for the recorded events, returns the summed device milliseconds and launch counts since
 * the last read (any pointer may be NULL), and resets the accumulators. */
int fftstencil_set_profiling(fftstencil_plan* plan, int enable);
int fftstencil_profile_read(fftstencil_plan* plan, double* fused_ms, int64_t* fused_launches,
                            double* band_ms, int64_t* band_launches);

/* Thread-local description of the last failure; "" after a successful call. */
const char* fftstencil_last_error(void);

/* ---- host-only introspection (no CUDA call; usable on a machine without a GPU) ----
 * Run the plan builder alone and report the geometry it would choose. */
int fftstencil_describe(int ndim, const int64_t* extents, const double* weights, int radius,
                        int T, fftstencil_info* info);

/* As fftstencil_describe with creation `flags`. */
int fftstencil_describe_ex(int ndim, const int64_t* extents, const double* weights, int radius, int T,
                           int flags, fftstencil_info* info);

/* Export the host plan's auxiliary tables, for tests of the plan builder:
 *   which = 0: forward DFT matrix of axis `axis` (1D: axis 0 -> F_N1, axis 1 -> F_N2;
 *              factored 2D plans: axis 0 -> F_8, axis 1 -> the twiddles w64^(ka*lb)),
 *              row-major complex as interleaved (re, im) pairs;
 *   which = 1: powered spectrum S_t (t = `t`, 1..T) in the kernel's order (2D:
 *              natural [k0][k1]; 3D: [k1][k2][k0]; 1D: N1 x N2 matrix in the Ruritanian
 *              order of Eq. 8),
 *              2*prod(tile) doubles (interleaved complex);
 *   which = 2: tile origins / ownership: for each tile (row-major tile order), per
 *              axis: origin, first owned cell, owned count -> 3*ndim*tiles int64
 *              values written as doubles.
 *   which = 3: 1D only: the prime-factor input map, N1*N2 entries: position l of the
 *              tile element stored at matrix cell (l1, l2) (row-major), as doubles.
 * `out` must hold `cap` doubles; returns the number of doubles needed (>= 0) or a
 * negative code.  Call with out = NULL to query the size. */
int64_t fftstencil_export_aux(int ndim, const int64_t* extents, const double* weights, int radius,
                              int T, int which, int axis, int t, double* out, int64_t cap);

/* Host-only: the op list fftstencil_run_host issues for a single-GPU plan of these arguments
 * with `chunks` = K and `depth` = Q (the FFTSTENCIL_E2E_PIPE / _DEPTH values), for tests of the
 * schedule.  4 int64 per op, in issue order:
 *   {0, y0, y1, 0}  copy input rows [y0, y1) host -> device, then the run stream waits for it;
 *   {1, y0, y1, 0}  copy the fixed ring's rows [y0, y1) into both pass buffers;
 *   {2, k, u0, u1}  pass k (1-based, t = T, the last pass total_steps mod T if nonzero) on
 *                   outer tile rows [u0, u1): their fused tile pairs and the band cells in
 *                   rows [row(u0), row(u1)), row(u) = 0 / u*S + h / n0 for u = 0 / inner / U;
 *   {3, y0, y1, 0}  copy result rows [y0, y1) device -> host after all earlier ops.
 * `out` must hold `cap` ops (4*cap int64); returns the number of ops (>= 0; out = NULL
 * queries it) or FFTSTENCIL_EINVAL when the plan does not take the pipelined path (1D,
 * h > S, fewer than 2*chunks outer tile rows, chunks < 2, depth < 1, total_steps <= 0). */
int64_t fftstencil_e2e_schedule(int ndim, const int64_t* extents, const double* weights, int radius,
                                int T, int64_t total_steps, int chunks, int depth, int64_t* out,
                                int64_t cap);

#ifdef __cplusplus
}
#endif

#endif /* FFTSTENCIL_H */
