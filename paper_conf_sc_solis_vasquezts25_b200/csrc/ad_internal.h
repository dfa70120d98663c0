// ad_internal.h — device-side data layout of libad (not part of the ABI).
//
// A ligand lives in ONE contiguous, 16-byte aligned blob that a CTA stages into
// shared memory with a single TMA bulk copy (cp.async.bulk) and keeps for all
// max_iters ADADELTA iterations.  Layout (offsets in LigHeader, bytes):
//
//   LigHeader                                   224 B
//   atoms   float4 [N]      reference x,y,z (A, DFS order), charge q
//   info    int2   [N]      {map | type<<8 | chain_len<<16 | slot<<24, chain_start}; slot =
//                           the atom's storage row in the per-pose X / gradient arrays
//   tors    float4 [T][2]   reference-frame axis point P_b and unit axis u_b
//   tors64  double [T][6]   the same in FP64 (u_b normalised in FP64), for the torsion chain
//   tinfo   int4   [T]      {a_b, c_b, lo_b, hi_b}: axis atoms (storage rows) and the moving set
//                           M_b = [lo_b, hi_b) (contiguous thanks to DFS order)
//   chain   u8     [Lrot]   per atom: the torsions moving it, leaf -> root
//   mask    u32x2  [N]      per atom bitmask of torsions moving it (baseline engine)
//   prec    u32    [R*64]   pair schedule: i | j<<8 | slot_i<<16 | slot_j<<20 | tp<<24
//                           (slot_i == K marks an empty place).  Step r holds entries
//                           [64r, 64r+64): lane l takes 64r+l and 64r+32+l; within a
//                           step every (slot, atom) target is distinct -> no atomics.
//   pdsv    f32x2  [R*64]   per pair (desolvation prefactor c_ds[(Si+Q|qi|)Vj+(Sj+Q|qj|)Vi],
//                           coeff_el q_i q_j), both rounded once from FP64
//           (INTRA_OWNER: prec/pdsv hold [E][32] directed entries a|b<<8|tp<<16|flags<<24
//            instead, plus comb int2 [N] (start, count) into combidx u16 [..] = the
//            partial slots k*32+lane that belong to atom a)
//   tp      float4 [nt*nt*8] cA, cB, r0, n (m == 12); 8 copies per entry (index t*8+c),
//                           lane l reads copy l%8 -> conflict-free 128-bit lookups
//   pka     u32x4  [R*32]   (cherry schedule, off_pk != 0: INTRA_SCATTER with the schedule
//   pkb     f32x4  [R*32]   in shared memory; R = n_rounds cherry steps of 32 lanes, each lane
//   pkc     f32x4  [R*32]   two pairs sharing a centre atom) -- see intra_cherry in ad_kernels.cuh;
//           global-memory cherries (PK_GMEM): pkc f32x2 [R*32] (40-B records, pack_cherries compact)
//           The warp engine stages the whole blob; the paper-style baseline stages
//           [0, off_pk) (prec / pdsv / tp), its footprint unchanged.
//
// Per-warp scratch (after the blob, one slice per warp), see WarpScratch below.
#pragma once
#include <cstdint>

namespace adk {

constexpr int kLanes = 32;
constexpr int kMaxGenes = 64;
constexpr int kPairsPerStep = 64;  // 2 pairs per lane per step of the intra loop

// indices into LigHdr::ff
enum {
    FF_DELTA = 0,     // smooth / 2
    FF_CUT_VDW = 1,
    FF_CUT_EL = 2,
    FF_EL_RMIN = 3,
    FF_DIEL_A = 4,
    FF_DIEL_B = 5,
    FF_DIEL_K = 6,
    FF_DIEL_LB = 7,   // lambda * B
    FF_COEFF_EL = 8,
    FF_DS_EXP2 = 9,   // -log2(e) / (2 sigma^2)
    FF_INV_S2 = 10,   // 1 / sigma^2
    FF_W_OUT = 11,
    FF_N = 16
};

// Intra-pair evaluation modes (chosen at upload, uniform per ligand):
//   INTRA_SCATTER: each pair evaluated once; steps of 64 pairs with distinct
//                  (slot, atom) gradient targets -> read-modify-write, __syncwarp per step.
//   INTRA_OWNER:   "owner computes": every pair evaluated from both ends (full
//                  contributor list, 2x pair flops); lane l walks a balanced slice
//                  of the atom-sorted directed list, accumulates g_a in registers and
//                  stores one partial per (lane, atom chunk); no scatter, no sync in
//                  the loop; partials are combined per atom afterwards.
//   INTRA_HYBRID:  every pair once; the owner side (i = min(i, j)) accumulates in
//                  registers along runs of equal owner, the partner side is a
//                  conflict-free read-modify-write as in INTRA_SCATTER (half the
//                  shared-memory RMW traffic, no duplicated flops).
enum { INTRA_SCATTER = 0, INTRA_OWNER = 1, INTRA_HYBRID = 2 };
// LigHeader.pk_flags: PK_GMEM = the cherry records stay in global memory (not staged;
// intra_cherry_gm, 128-register kernels); PK_PRED = empty ends share dummy gradient
// rows with other lanes of their step, so their stores are predicated off (else every
// dummy target of a step is a distinct row and the loop stores unconditionally).
enum { PK_GMEM = 1, PK_PRED = 2 };
// owner-mode entry: a | b<<8 | tp<<16 | flags<<24
enum { OF_PRIMARY = 1, OF_FIRST = 2, OF_LAST = 4, OF_DUMMY = 8 };

struct alignas(16) LigHeader {
    int32_t n_atoms, n_tors, n_pairs, n_types;          // 16
    int32_t n_rounds, n_slots, n_chain, blob_bytes;     // 32
    int32_t off_atoms, off_info, off_tors, off_tinfo;   // 48
    int32_t off_chain, off_mask, off_prec, off_pdsv;    // 64
    int32_t off_tp, scratch_bytes, n_pad, intra_mode;   // 80
    int32_t n_entries, n_chunks, off_comb, off_combidx; // 96  (owner mode: E per lane, chunks per lane)
    int32_t pairs_gmem, stage_bytes, ws_g, ws_w;        // 112: schedule in global memory?, bytes staged to smem
    int32_t ws_d, ws_trig, ws_tw, ws_genes;             // 128  per-warp scratch offsets (WarpScratch, ws_x = 0),
    int32_t ws_part, off_pk, base_rounds, base_slots;   // 144  precomputed so kernels reload, not recompute, them;
                                                        //      off_pk: cherry records (0 = none); base_*: steps
                                                        //      and slots of the prec list (= n_rounds / n_slots
                                                        //      unless the warp engine runs a cherry schedule)
    int32_t off_pkg, off_tors64, ws_trig64, pk_flags;   // 160  off_pkg: pre-decoded global-memory places (0 = none);
                                                        //      off_tors64: double [T][6] axis point P_b, unit axis u_b
                                                        //      (the FP64 torsion chain); ws_trig64: per-warp double2 [T];
                                                        //      pk_flags (PK_*): how the cherry loop runs
    float ff[FF_N];                                     // 224
};
static_assert(sizeof(LigHeader) == 224, "header size");

// Device table entry, one per uploaded ligand.
struct LigDev {
    const unsigned char* blob;  // global copy of the whole blob
    int32_t blob_bytes;         // bytes the warp engine stages into shared memory (header .. tables [.. schedule])
    int32_t scratch_bytes;      // per-warp scratch, TC engine
    int32_t scratch_simt;       // per-warp scratch, SIMT engine (no D tile)
    int32_t base_bytes;         // bytes the paper-style baseline stages from base_blob
    const unsigned char* base_blob;  // the baseline's blob (== blob unless the warp engine runs cherries)
};

// Grid in device memory, x-pair layout:
//   tmap [n_type][nz][ny][nx] float2 (v[x], v[x+1])
//   ed   [nz][ny][nx]         float4 (E[x], E[x+1], D[x], D[x+1])
// Cell-record layout (layout == 1, used when it fits comfortably in L2): for every
// cell (x,y,z) the 8 corner values, corner index dx + 2 dy + 4 dz:
//   tc8 [n_type][nz][ny][nx][8]  (32 B, one 256-bit load per atom)
//   ed8 [nz][ny][nx][16]         (E corners then D corners, 64 B, two 256-bit loads)
// -> 3 loads / 96 B per atom = the algorithmic bytes, 8x the map memory.
struct GridDev {
    const float2* tmap;
    const float4* ed;
    const float* tc8;
    const float* ed8;
    int32_t nx, ny, nz, n_type;
    float ox, oy, oz, h, inv_h;
    int32_t layout;  // 0 = x-pair, 1 = cell records
};

// Per-warp scratch layout (offsets in bytes from the warp's slice; 16-aligned).
struct WarpScratch {
    int32_t x;      // float4 [Npad+8]      world coords + charge (+ 8 zero-charge rows)
    int32_t g;      // float4 [K][Npad]+8   atom gradient accumulators (slot 0 seeded with inter) + 8 spare
    int32_t w;      // float4 [Npad+1][2]   W staging (TC engines only)
    int32_t d;      // float  [Mpad][8]     D = M_ext W (TC)
    int32_t trig;   // float2 [T+3]         cos, sin of torsion angles, then phi, theta, alpha/2
    int32_t trig64; // double2 [T]          sin, 1 - cos of torsion angles in FP64 (the chain)
    int32_t tw;     // float4 [6 + T][2]    per-gene gradient vectors U_k, W_k (.w: sum rows)
    int32_t genes;  // float  [64]
    int32_t part;   // float4 [C][32]       owner mode: per-(lane, chunk) partial gradients
    int32_t bytes_simt;
    int32_t bytes;
};

__host__ __device__ inline int32_t align16(int32_t v) { return (v + 15) & ~15; }

__host__ __device__ inline WarpScratch warp_scratch_layout(int32_t n_atoms, int32_t n_tors, int32_t n_slots,
                                                           int32_t n_chunks, int32_t n_spare = 8) {
    WarpScratch s;
    const int32_t npad = (n_atoms + 7) & ~7;
    const int32_t mpad = (n_tors + 1 + 15) / 16 * 16;
    int32_t o = 0;
    // X rows + 8 zero-charge rows (positions (r,0,0), bank group r) that the empty
    // ends of cherry schedules read
    s.x = o;     o += 16 * (npad + 8);
    // rows of npad float4 (slot k of atom a at k * npad + a) + n_spare spare rows
    // K * npad + (0..n_spare-1): the targets of empty schedule places (8, or the
    // distinct dummy rows of a cherry schedule without PK_PRED)
    s.g = o;     o += 16 * npad * n_slots + 16 * n_spare;
    s.trig = o;  o += align16(8 * (n_tors + 3));  // torsions, then phi, theta, alpha/2
    s.trig64 = o; o += 16 * n_tors;
    s.tw = o;    o += 32 * (6 + n_tors);  // per-gene gradient vectors (U, W) + rows
    s.genes = o; o += 4 * kMaxGenes;
    // right after the genes, narrow ligands (6 + T <= 32, one gene per lane): the per-lane
    // ADADELTA state between updates (float4: E[g^2], E[dx^2], best gene, best E)
    if (6 + n_tors <= 32) o += 16 * 32;
    s.part = o;  o += 16 * 32 * n_chunks;
    // the SIMT engine needs neither W nor D: its prefix sums overwrite the X and
    // slot-0 gradient rows the scan has just consumed (ad_kernels.cuh, a4-a5), so
    // its per-warp footprint ends here (a smaller shared-memory carve-out leaves
    // more L1 for the grid gathers)
    s.bytes_simt = o;
    s.w = o;     o += 32 * (npad + 1);              // TC engines: W staging
    s.d = o;     o += align16(4 * 8 * mpad);
    s.bytes = o;
    return s;
}

// Baseline engine (one block per pose) shared-memory layout after the blob.
struct BlockScratch {
    int32_t x, g, trig, trig64, tw, tacc, red, genes, stage, bytes;
};

// stage: [stage_threads][8] floats for the TCEC variant's tensor-core reduction
// (0 for the SIMT baseline, so its footprint is not inflated)
__host__ __device__ inline BlockScratch block_scratch_layout(int32_t n_atoms, int32_t n_tors, int32_t stage_threads) {
    BlockScratch s;
    int32_t o = 0;
    const int32_t t1 = n_tors > 0 ? n_tors : 1;
    const int32_t npad = (n_atoms + 7) & ~7;  // rows are storage slots (< npad)
    s.x = o;     o += 16 * npad;
    s.g = o;     o += 16 * npad;
    s.trig = o;  o += align16(8 * (n_tors + 3));
    s.trig64 = o; o += 16 * t1;
    s.tw = o;    o += 32 * t1;
    s.tacc = o;  o += align16(4 * t1);
    s.red = o;   o += 4 * 16;
    s.genes = o; o += 4 * kMaxGenes;
    s.stage = o; o += 32 * stage_threads;
    s.bytes = o;
    return s;
}

// Scoring constants of the pair term and the out-of-grid weight, derived from a
// ligand's LigHeader::ff on the host and passed as kernel parameters: the kernels
// use them as constant-bank operands, so they occupy no registers in the pair loop.
// Every ligand of one launch must share them (ad_api.cu checks on the host).
struct PairConst {
    float delta, cut_vdw, cut_el, rmin, A, B, k, nlB2, kBlB, coeff_el, ds_exp2, inv_s2, w_out;
};

__host__ __device__ inline PairConst pair_const_from_ff(const float* ff) {
    PairConst c;
    c.delta = ff[FF_DELTA];
    c.cut_vdw = ff[FF_CUT_VDW];
    c.cut_el = ff[FF_CUT_EL];
    c.rmin = ff[FF_EL_RMIN];
    c.A = ff[FF_DIEL_A];
    c.B = ff[FF_DIEL_B];
    c.k = ff[FF_DIEL_K];
    c.nlB2 = -ff[FF_DIEL_LB] * 1.4426950408889634f;  // exp(-lB r) = ex2(nlB2 r)
    c.kBlB = ff[FF_DIEL_K] * ff[FF_DIEL_B] * ff[FF_DIEL_LB];
    c.coeff_el = ff[FF_COEFF_EL];
    c.ds_exp2 = ff[FF_DS_EXP2];
    c.inv_s2 = ff[FF_INV_S2];
    c.w_out = ff[FF_W_OUT];
    return c;
}

struct KParams {
    GridDev grid;
    PairConst pc;
    const LigDev* ligs;
    int32_t lig;
    const int32_t* pose_ligand;
    int32_t n_poses;
    int32_t stride;
    float* genes;
    float* energy;
    float* grad;
    float* aux;
    float* trace;
    int64_t* n_evals;
    int32_t* err;        // device error word (ERR_* bits, atomicOr)
    int32_t* err_seen;   // mapped pinned host word: set on the (rare) error path only
    int32_t max_iters;
    float rho, eps;
    int32_t smem_blob;      // bytes reserved for the blob in shared memory
    int32_t smem_scratch;   // bytes per warp (SIMT/TC) or per block (baseline)
    int32_t n_ligs;
    const int32_t* n_active;  // optional device count: poses >= *n_active exit (LGA's compacted LS list)
    int64_t* phase_cycles;    // A14 instrumented kernels only: [n_poses][PH_N] clock64 cycles per phase
};

// A14 phases (ad_ls_params.phase_cycles): indices of the per-pose cycle counters
enum Phase { PH_POSE_INTER = 0, PH_INTRA = 1, PH_ASSEMBLE = 2, PH_REDUCE = 3, PH_UPDATE = 4, PH_N = 5 };

// NEXT-3 GA generation parameters (ad_lga_params minus the LS part)
struct GaParams {
    int32_t pop, n_genes, stride, elitism;
    float cross_rate, mut_rate, tour_rate, ls_rate, dmov, dang;
    uint64_t seed;
};

// device error bits
enum { ERR_BAD_LIGAND = 1, ERR_FOOTPRINT = 2, ERR_MIXED_CTA = 4, ERR_STRIDE = 8 };

}  // namespace adk
