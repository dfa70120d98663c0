/*
 * ad.h — C ABI of libad: the B200 (sm_100a) ADADELTA energy+gradient hot path
 * of AutoDock-GPU as described in Solis-Vasquez et al., "Architecting Tensor
 * Core-Based Reductions for Irregular Molecular Docking Kernels" (IA3 @ SC'25).
 *
 * Citations: P:Ln = /root/reference/PAPER.md line n.  Readings Z-k / O-k are
 * the ones listed in DESIGN.md (originally SURVEY.md §8(c)).
 *
 * Conventions (all entry points):
 *   - Every function returns an ad_status (int32): AD_OK = 0, negative = error.
 *     No C++ exception, abort or exit crosses the ABI.  ad_last_error() returns
 *     a thread-local, human-readable message for the last failing call.
 *   - Host pointers are read during the call and never retained.  Device
 *     pointers (pose, output and trace buffers) are caller-owned; the library
 *     only reads/writes them from kernels enqueued on `cuda_stream`.
 *   - `cuda_stream` is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  Compute calls enqueue asynchronously and return; a kernel fault
 *     surfaces as AD_ERR_CUDA on a later call or stream synchronisation.
 *     Device-side argument errors (bad pose_ligand ids) surface as
 *     AD_ERR_INVALID_ARG on a later call on the same context once the
 *     offending kernel has completed (no call blocks to find out), or at
 *     ad_sync().
 *   - One context per device per host thread, except ad_upload_ligand and
 *     ad_free_ligand, which may be called concurrently from several host threads
 *     on one context (the host-side ligand preparation -- torsion tree, pair
 *     schedule -- runs unlocked, so a screen's uploads overlap; the device-side
 *     part is serialised internally).
 *   - Units: Angstrom, kcal/mol, elementary charge, degrees (Z11).
 */
#ifndef AD_H
#define AD_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

enum ad_status {
    AD_OK = 0,
    AD_ERR_INVALID_ARG = -1, /* null/inconsistent argument, index out of range */
    AD_ERR_LIMIT = -2,       /* size beyond the compile-time limits below */
    AD_ERR_CUDA = -3,        /* CUDA runtime error (message in ad_last_error) */
    AD_ERR_OOM = -4,         /* device allocation failed */
    AD_ERR_STATE = -5        /* call order violated (e.g. no grids uploaded) */
};

enum ad_engine {
    /* Warp-per-pose kernel, gene-space sums by a warp prefix scan over atoms
     * in torsion-tree DFS order (FP32 shuffles, no block barrier). */
    AD_ENGINE_SIMT = 0,
    /* Same kernel, gene-space sums D = M_ext * W as error-corrected TF32
     * tensor-core MMAs (mma.sync m16n8k8; hi/lo split of W, accumulation
     * outside the tensor core in FP32 round-to-nearest: P:L186-199). */
    AD_ENGINE_TC = 1,
    /* Paper-style baseline: one thread block per pose, 7 sequential
     * block-level sum reductions per gradient plus
     * shared-memory atomics, all on FP32 SIMT cores.  The speedup denominator. */
    AD_ENGINE_PAPER_BASELINE = 2,
    /* The same block-per-pose kernel with the seven reductions replaced by one
     * tensor-core reduction of all seven values (ones-row MMA, Eq 1 generalised)
     * with the TF32 hi/lo error correction: the paper's TCEC in its
     * own design context (local search only). */
    AD_ENGINE_PAPER_TCEC = 3,
    /* NEXT-2 accuracy study: the warp-per-pose kernel with every sum (energy and
     * D = M_ext * W) on the tensor cores in FP16 WITHOUT error correction: FP16
     * operands and an FP16 accumulator kept inside the tensor core across
     * k-steps (mma.sync m16n8k16 .f16.f16.f16.f16) -- the Schieffer-Peng
     * reduction the paper starts from (Lst 1 bottom), whose
     * accuracy loss (Fig 1) motivates TCEC.  Not for production use. */
    AD_ENGINE_TC_FP16 = 4
};

/* Compile-time limits (violations return AD_ERR_LIMIT). */
#define AD_MAX_ATOMS 256   /* u8 atom indices in the pair schedule */
#define AD_MAX_TORS 58     /* 6 + 58 = 64 genes; AD-GPU supports 57 */
#define AD_MAX_TYPES 32
#define AD_MAX_MAPS 34     /* n_type_maps + electrostatic + desolvation */
#define AD_MAX_LIGANDS 65536

typedef struct ad_context ad_context;
typedef int32_t ad_ligand_id;

/* Thread-local message of the last failing call ("" if none). */
const char* ad_last_error(void);

/* Library ABI version (increments on incompatible changes). */
int32_t ad_version(void);

/* Create a context bound to CUDA device `cuda_device`.  *out receives the
 * handle (NULL on failure).  Errors: AD_ERR_INVALID_ARG (out NULL / bad
 * device), AD_ERR_CUDA. */
int32_t ad_context_create(int32_t cuda_device, ad_context** out);

/* Release every device buffer of the context (grids, ligands).  Synchronises
 * the device first.  NULL is accepted (no-op). */
int32_t ad_context_destroy(ad_context* ctx);

/* Receptor grid maps (D3; AutoGrid maps listed by
 * protein.maps.fld).  Grid point (i,j,k) sits at origin + spacing*(i,j,k);
 * maps are [n_maps][nz][ny][nx], x fastest.  Maps 0..n_maps-3 are per-atom-type
 * affinity maps, n_maps-2 the electrostatic map (multiplied by the atom
 * charge q), n_maps-1 the desolvation map (multiplied by |q|).  O-2, Z5, Z20. */
typedef struct {
    int32_t nx, ny, nz; /* grid points per axis (>= 2 each) */
    int32_t n_maps;     /* 3..AD_MAX_MAPS */
    float spacing;      /* A, > 0 */
    float origin[3];    /* A, position of grid point (0,0,0) */
} ad_grid_desc;

/* Copy the maps into library-owned device memory, re-laid out for the
 * kernels' gathers (x-pair records, elec/desolv interleaved).
 * `maps` is a host pointer, or a device pointer if maps_on_device != 0.
 * Replaces any previous grid of the context.  Enqueued on `cuda_stream`; the
 * caller may reuse `maps` when the call returns for host maps (copied
 * synchronously), or after the stream completes for device maps.
 * Errors: AD_ERR_INVALID_ARG, AD_ERR_LIMIT, AD_ERR_OOM, AD_ERR_CUDA. */
int32_t ad_upload_grids(ad_context* ctx, const ad_grid_desc* desc, const float* maps, int32_t maps_on_device,
                        void* cuda_stream);

/* Scoring-function constants (O-2, O-3; AutoDock4.2 defaults in DESIGN.md). */
typedef struct {
    float smooth;        /* A, width of the flat band around r0 (delta = smooth/2), Z6 */
    float cut_vdw;       /* A, vdW / H-bond cutoff (strict <), Z7 */
    float cut_el;        /* A, electrostatics / desolvation cutoff (strict <), Z7 */
    float el_rmin;       /* A, floor on r in the electrostatic term, Z8 */
    float diel_A, diel_B, diel_k, diel_lambda; /* eps(r) = A + B / (1 + k exp(-lambda B r)) */
    float coeff_el;      /* kcal/mol A / e^2 (332.06363 x FE_coeff_estat) */
    float coeff_ds;      /* FE_coeff_desolv */
    float qasp;          /* charge-dependent desolvation factor Q */
    float sigma_ds;      /* A, desolvation Gaussian width */
    float w_out;         /* kcal/mol per (grid unit)^2, out-of-grid restraint, Z4 */
} ad_ff_params;

/* Ligand (D4-D7).  All pointers are HOST pointers, read and copied
 * during ad_upload_ligand.  The library renumbers atoms internally (torsion-
 * tree DFS order) and builds its own pose chains and pair schedule; outputs are
 * in gene space only, so the renumbering is invisible to callers. */
typedef struct {
    int32_t n_atoms;            /* 1..AD_MAX_ATOMS */
    int32_t n_tors;             /* 0..AD_MAX_TORS */
    int32_t n_pairs;            /* >= 0 */
    int32_t n_types;            /* 1..AD_MAX_TYPES */
    const float* ref_xyz;       /* [n_atoms][3] A, rotation centre at the origin (Z22) */
    const int32_t* atom_map;    /* [n_atoms] type-map index 0..n_maps-3 */
    const int32_t* atom_type;   /* [n_atoms] intra type 0..n_types-1 */
    const float* charge;        /* [n_atoms] e */
    const int32_t* tors_axis;   /* [n_tors][2] (a fixed side, c moving side), listed root -> leaf (Z13) */
    const uint8_t* tors_moving; /* [n_tors][n_atoms] 0/1; moving sets must be nested or disjoint
                                   (a rotatable-bond tree), a not in its own set, c in it */
    const int32_t* pairs;       /* [n_pairs][2] intramolecular contributors, i != j (Z9) */
    const float* tp_coef;       /* [n_types][n_types][5] cA, cB, r0, m, n with m == 12 and
                                   n in {6, 10} (12-6 vdW / 12-10 H-bond, Z10) */
    const float* type_S;        /* [n_types] desolvation solvation parameter S */
    const float* type_V;        /* [n_types] desolvation volume V */
    const ad_ff_params* ff;     /* scoring constants for this ligand */
} ad_ligand_desc;

/* Upload a ligand; *out receives its id (>= 0; the lowest id not in use, so ids
 * of freed ligands are reused).  Requires a grid (atom_map must index a type
 * map).  Thread-safe with respect to other uploads / frees on the same context.
 * Errors: AD_ERR_INVALID_ARG (bad index, a not excluded from its moving set,
 * non-laminar moving sets, i == j pair, unsupported exponents), AD_ERR_LIMIT,
 * AD_ERR_STATE (no grid), AD_ERR_OOM. */
int32_t ad_upload_ligand(ad_context* ctx, const ad_ligand_desc* desc, ad_ligand_id* out);

/* Free a ligand's device blob (synchronises the device). */
int32_t ad_free_ligand(ad_context* ctx, ad_ligand_id lig);

/* Launch set of later pose_ligand launches (ad_score_poses, ad_local_search,
 * ad_lga_run with pose_ligand != NULL): the ligands they may reference, which
 * size their shared memory, pick the >32-gene variant and must share one
 * ad_ff_params.  ids: host [n] live ligand ids, copied; n == 0 restores the
 * default (every live ligand).  A launch that references a ligand whose
 * footprint exceeds the set's fails with AD_ERR_INVALID_ARG on the next call
 * (device-side check).  A virtual screen keeps all its ligands resident and
 * sets each bucket's ligands before the bucket's launch.
 * Errors: AD_ERR_INVALID_ARG (an id not live). */
int32_t ad_set_launch_ligands(ad_context* ctx, const int32_t* ids, int32_t n);

/* Host effort of later uploads' intra-pair schedule placement (DESIGN.md §7,
 * "Bank-conflict-free placement"): 2 (default) = full search (1-500 ms of host
 * time per ligand, conflict-free shared-memory accesses); 1 = a tenth of the
 * local-search iterations; 0 = construction only (no cross-step rebalancing,
 * no local search; ~1 ms).  Every effort evaluates the same pairs with the same
 * arithmetic; only the order of the intra-pair partial sums (FP32 rounding, well
 * inside the parity gates) and the kernel's shared-memory bank conflicts
 * (speed) change.  Errors: AD_ERR_INVALID_ARG. */
int32_t ad_set_schedule_effort(ad_context* ctx, int32_t effort);

/* One energy (+ gradient) evaluation per pose: PoseCalculation -> InterGradient
 * -> IntraGradient -> gene-space sums (Alg 4; energy = inter + intra,
 * O-5).  One warp per pose.
 *   lig          ligand of every pose (if pose_ligand == NULL).
 *   pose_ligand  device [n_poses] ligand ids, or NULL.  Shared memory is then
 *                sized for the largest ligand of the launch set (every live
 *                ligand, or the list given to ad_set_launch_ligands), and every
 *                aligned group of poses sharing a CTA must use one ligand (groups
 *                of 1, 2, 4 or 8 poses; keep runs of one ligand a multiple of 8
 *                poses long).
 *   genes        device [n_poses][geno_stride] FP32, geno_stride >= 6 + n_tors:
 *                translation (grid units), phi, theta, alpha, torsions (degrees).
 *   energy       device [n_poses] FP32 out.
 *   grad         device [n_poses][geno_stride] FP32 out (dE/dgene, padding
 *                columns untouched), or NULL for energy only (NEXT-1).
 *   aux          device [n_poses][8] FP32 out or NULL: E_inter, E_intra,
 *                torque xyz (kcal/mol), sum of atom gradients xyz (kcal/mol/A).
 * n_poses == 0 is a no-op.  Errors: AD_ERR_INVALID_ARG, AD_ERR_STATE,
 * AD_ERR_CUDA. */
int32_t ad_score_poses(ad_context* ctx, ad_ligand_id lig, const int32_t* pose_ligand, int32_t n_poses,
                       const float* genes, int32_t geno_stride, float* energy, float* grad, float* aux,
                       void* cuda_stream);

/* ADADELTA local-search parameters (Alg 3; Zeiler [19] P:L406). */
typedef struct {
    int32_t max_iters;      /* evaluations per pose (default 300); >= 1 */
    float rho, eps;         /* decay and conditioning constants (0.8, 0.01; Z14) */
    int32_t pop_per_run;    /* poses per run for run_best; 0 = no run_best */
    int32_t engine;         /* enum ad_engine */
    int32_t warps_per_cta;  /* poses per CTA for SIMT/TC/TC_FP16, 0..32 (0 = library choice);
                               threads per block for PAPER_BASELINE (0 = 64) */
    float* trace;           /* optional device [n_poses][max_iters][1 + 2*geno_stride]:
                               per evaluation E, genes, gradient (Z19 shadowed parity) */
    int64_t* phase_cycles;  /* optional device [n_poses][5] (A14 instrumentation):
                               clock64 cycles per pose summed over the iterations, spent in
                               (0) pose + inter, (1) intra pairs, (2) gradient assembly
                               (per-atom gradients, torques, gene gradients from the sums),
                               (3) reductions (energy sum + the gene-space sums proper),
                               (4) update (best tracking, ADADELTA).  Non-NULL runs a
                               separately compiled instrumented kernel (SIMT, TC and the
                               paper-style engines; AD_ERR_INVALID_ARG for TC_FP16).  The
                               paper's reduction fraction is f = (3) / total.  Ignored by
                               ad_lga_run. */
} ad_ls_params;

/* ADADELTA local search, one pose per warp (or per block for
 * PAPER_BASELINE), max_iters evaluations each.  With pose_ligand != NULL and
 * pop_per_run > 0 every run (pop_per_run consecutive poses) must belong to one
 * ligand; CTA groups are then sized to divide pop_per_run (any population size
 * works).  Per pose: evaluate (E, grad) of the
 * current genotype, keep it if E < best (strict; earliest wins), update every
 * gene (Z15, Z16: no angle wrapping).  On return (stream order):
 *   genes        in: start genotypes; out: best genotype per pose.
 *   best_energy  device [n_poses] FP32 best energy.
 *   run_best     device [n_poses/pop_per_run][1 + geno_stride] FP32 or NULL:
 *                per run the lowest best_energy (ties -> lowest pose index)
 *                followed by that pose's genes (O-8); columns past
 *                6 + n_tors are 0 (single ligand) or the pose row's padding
 *                (pose_ligand != NULL).  Requires n_poses % pop_per_run == 0.
 *   n_evals      device int64 accumulator or NULL; += n_poses * max_iters.
 * Errors: AD_ERR_INVALID_ARG, AD_ERR_STATE, AD_ERR_CUDA. */
int32_t ad_local_search(ad_context* ctx, ad_ligand_id lig, const int32_t* pose_ligand, int32_t n_poses,
                        float* genes, int32_t geno_stride, float* best_energy, float* run_best, int64_t* n_evals,
                        const ad_ls_params* params, void* cuda_stream);

/* NEXT-3: the Lamarckian GA around the local search (Alg 1).
 * n_runs independent runs (coarse level) of pop_size individuals.  Each
 * generation of an unfinished run: GA(population) -- elitism, binary tournaments
 * (the better of two random individuals wins with probability tour_rate),
 * two-point crossover (probability cross_rate), per-gene uniform mutation
 * (probability mut_rate; +-dmov grid units on translation genes, +-dang degrees
 * on angle genes) -- then the energy of every new individual, then
 * LS(population): each individual with probability ls_rate runs ADADELTA
 * (`ls`) and is replaced by its best genotype (Lamarckian).  A run
 * stops when its evaluation count (pop per generation + LS individuals x
 * ls.max_iters) reaches max_evals or its generation count reaches max_gens
 * (2 500 000 and 27 000).  The operator parameters are not in the
 * paper (DESIGN.md §7b readings; AutoDock-GPU defaults).  Random numbers: a
 * counter-based SplitMix64 chain per (seed, generation, run, individual, draw),
 * so results do not depend on launch shapes.
 *   genes      device [n_runs * pop_size][geno_stride]: in = initial population,
 *              out = final population (caller-owned)
 *   energies   device [n_runs * pop_size]: out, final energies
 *   run_best   device [n_runs][1 + geno_stride] or NULL: best energy + genes per run
 *   n_evals    device int64 [n_runs] or NULL: evaluations per run
 *   n_gens     device int32 [n_runs] or NULL: generations per run
 * Blocks the calling thread until every run finished (one 4-byte read per
 * generation); scratch is allocated per call.  Engines: SIMT, TC, TC_FP16. */
typedef struct {
    int32_t pop_size;       /* individuals per run (150) */
    int32_t max_gens;       /* N_gens^MAX (27000) */
    int64_t max_evals;      /* N_score-evals^MAX per run (2 500 000) */
    int32_t elitism;        /* best individuals copied unchanged (1) */
    float cross_rate;       /* 0.8 */
    float mut_rate;         /* 0.02 per gene */
    float tour_rate;        /* 0.6 */
    float ls_rate;          /* 0.8 */
    float dmov;             /* mutation half-width, translation genes, grid units */
    float dang;             /* mutation half-width, angle genes, degrees (90) */
    uint64_t seed;
    ad_ls_params ls;        /* the local search (pop_per_run and trace ignored) */
} ad_lga_params;

int32_t ad_lga_run(ad_context* ctx, ad_ligand_id lig, int32_t n_runs, float* genes, int32_t geno_stride,
                   float* energies, float* run_best, int64_t* n_evals, int32_t* n_gens, const ad_lga_params* params,
                   void* cuda_stream);

/* Reduction-engine microbenchmark (config 4; Eq 1-5): sum each of
 * n_comp components over n_partials per block.
 *   partials  device [n_blocks][n_partials][n_comp] FP32
 *   out       device [n_blocks][n_comp] FP32
 *   engine    AD_ENGINE_SIMT (warp transpose-butterfly + one smem exchange),
 *             AD_ENGINE_TC (ones-vector TF32 MMA, hi/lo split, RN accumulation
 *             outside the tensor core), AD_ENGINE_PAPER_BASELINE (n_comp
 *             sequential block reductions with barriers), AD_ENGINE_TC_FP16
 *             (ones-vector FP16 MMA with the FP16 accumulator inside the tensor
 *             core, per-warp results combined in FP16: no EC, NEXT-2).
 * n_partials in {32, 64, ..., 1024} (multiple of 32), n_comp in 1..64. */
int32_t ad_reduce_blocks(ad_context* ctx, int32_t engine, int32_t n_blocks, int32_t n_partials, int32_t n_comp,
                         const float* partials, float* out, void* cuda_stream);

/* Wait for `cuda_stream` and report any device-side argument error recorded by
 * kernels enqueued so far (bad pose_ligand ids, a ligand outside the launch
 * set's footprint, CTA groups mixing ligands, a ligand with more genes than
 * geno_stride): AD_ERR_INVALID_ARG with the reasons in ad_last_error(), then
 * the error word is cleared.  Compute calls never block for this: they report
 * an error word once the work that set it has completed.  AD_ERR_CUDA for a
 * kernel fault. */
int32_t ad_sync(ad_context* ctx, void* cuda_stream);

/* Device properties useful to callers: number of SMs and the shared memory
 * footprint (bytes) the SIMT/TC kernel uses per pose for ligand `lig`. */
int32_t ad_query(ad_context* ctx, ad_ligand_id lig, int32_t* n_sms, int32_t* smem_per_pose, int32_t* blob_bytes);

/* Launch shape of the last hot-path kernel enqueued on this context (for
 * reporting): grid (CTAs), threads per CTA, dynamic shared memory bytes. */
int32_t ad_last_launch(ad_context* ctx, int32_t* grid, int32_t* block, int32_t* smem_bytes);

#ifdef __cplusplus
}
#endif

#endif /* AD_H */
