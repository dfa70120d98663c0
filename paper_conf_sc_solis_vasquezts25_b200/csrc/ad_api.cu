// ad_api.cu — host side of libad: the C ABI declared in include/ad.h.
//
// Upload-time preprocessing turns the paper's inputs (receptor maps, ligand
// with rotation list and intramolecular contributor list) into
// the device layouts of ad_internal.h:
//   * grids  -> x-pair records (type maps) and interleaved elec/desolv records,
//   * ligand -> torsion-tree DFS renumbering (every moving set contiguous),
//               per-atom leaf->root torsion chains with reference-frame axes,
//               a conflict-free pair schedule (rounds of 32, K gradient slots),
//               per-pair desolvation prefactors, (cA, cB, r0, n) table.
// Launches pick warps-per-CTA from the occupancy calculator.
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>  // header-only NVTX v3: ranges cost a pointer check unless a tool is attached

#include <algorithm>
#include <array>
#include <atomic>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <mutex>
#include <thread>
#include <vector>

#include "ad.h"
#include "ad_internal.h"
#include "ad_kernels.cuh"

namespace {
// NVTX range over one ABI call (Nsight Systems / Compute timelines; SURVEY §5 tracing)
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange&) = delete;
    NvtxRange& operator=(const NvtxRange&) = delete;
};
}  // namespace

using namespace adk;

namespace {

thread_local std::string g_err;

int32_t fail(int32_t code, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

#define CUDA_TRY(expr)                                                                          \
    do {                                                                                        \
        cudaError_t e_ = (expr);                                                                \
        if (e_ != cudaSuccess) {                                                                \
            return fail(e_ == cudaErrorMemoryAllocation ? AD_ERR_OOM : AD_ERR_CUDA, "%s: %s (%s:%d)", \
                        #expr, cudaGetErrorString(e_), __FILE__, __LINE__);                    \
        }                                                                                       \
    } while (0)

struct LigSlot {
    unsigned char* d_blob = nullptr;  // the warp engines' blob
    unsigned char* d_base = nullptr;  // the paper-style baseline's (== d_blob unless cherries)
    int32_t blob_bytes = 0;      // staged by the warp engine
    int32_t base_bytes = 0;      // staged by the paper-style baseline
    int32_t scratch_bytes = 0;   // per warp (TC engine)
    int32_t scratch_simt = 0;    // per warp (SIMT engine)
    int32_t block_scratch = 0;   // per block (baseline)
    int32_t n_atoms = 0, n_tors = 0;
    bool pkg = false;            // pre-decoded global-memory schedule (wide 128-register kernels)
    bool smem_cherry = false;    // shared-memory cherries without PK_PRED: the cherry-only kernels (CH = 1) run it
    bool gm_cherry = false;      // global-memory cherries: the CH = 2 kernels run it
    float ff[FF_N] = {};         // LigHeader::ff (kernel parameters of every launch)
    bool live = false;
};

}  // namespace

struct ad_context {
    int device = 0;
    int n_sms = 0;
    int max_smem_optin = 0;
    int smem_per_sm = 0;
    bool has_grid = false;
    GridDev grid{};
    int32_t grid_n_type = 0;
    void* d_tmap = nullptr;
    void* d_ed = nullptr;
    std::vector<LigSlot> ligs;
    LigDev* d_ligtab = nullptr;
    int32_t ligtab_cap = 0;
    int32_t* d_err = nullptr;
    // device error word: kernels atomicOr their ERR_* bits into d_err (device memory)
    // and, on that rare path only, store the bits they saw into h_err, a mapped pinned
    // host word (d_err_seen is its device address).  After every call an event is
    // recorded on the caller's stream; a later call reads h_err once the event has
    // completed -- no copy and no host-device synchronisation on the normal path --
    // and, if it is set, copies the complete d_err synchronously and reports it.
    int32_t* h_err = nullptr;
    int32_t* d_err_seen = nullptr;
    cudaEvent_t err_ev = nullptr;
    bool err_pending = false;
    // launch-shape caches: cudaFuncSetAttribute once per kernel, occupancy per
    // (kernel, threads, dynamic shared memory)
    std::mutex launch_mu;
    // launch_warp decisions: key (kernels, footprint, n_poses, request) -> (W, kernel, smem)
    struct LaunchKey {
        const void *lo, *hi;
        int32_t blob, scratch, n_poses, req, mixed, align, pkg;
        bool operator==(const LaunchKey& o) const {
            return lo == o.lo && hi == o.hi && blob == o.blob && scratch == o.scratch && n_poses == o.n_poses &&
                   req == o.req && mixed == o.mixed && align == o.align && pkg == o.pkg;
        }
    };
    struct LaunchPick {
        LaunchKey key;
        int w;
        const void* k;
        size_t smem;
    };
    std::vector<LaunchPick> launch_cache;
    std::vector<const void*> smem_opted;
    std::vector<std::array<long long, 4>> occ;  // {kernel, threads, smem, blocks}
    // AD_INTRA_MODE=owner|scatter at context creation (tuning knob; scatter measured
    // faster on config 2: 1.40e8 vs 1.26e8 evals/s, profiles/README.md)
    int intra_mode = INTRA_SCATTER;
    int32_t last_grid = 0, last_block = 0, last_smem = 0, last_maxreg = 0;
    // pair schedules above this size are read from global memory (AD_PAIRS_SMEM_MAX)
    int32_t pairs_smem_max = 16384;
    int32_t pk_smem_max = 32768;  // cherry-schedule record bytes (48 per lane-step) staged per CTA at most
    // host effort spent on the pair schedule's bank-conflict placement (ad_set_schedule_effort)
    int32_t sched_effort = 2;
    // ligands that pose_ligand launches may reference (ad_set_launch_ligands; empty = every
    // live ligand): shared memory, the wide variant and the common-constants check follow it
    std::vector<int> launch_set;
    // serialises the device-side part of ad_upload_ligand / ad_free_ligand (the host-side
    // ligand preparation runs outside it, so uploads from several threads overlap)
    std::mutex mu;
};

namespace {

int32_t set_device(ad_context* ctx) {
    int cur = -1;
    if (cudaGetDevice(&cur) == cudaSuccess && cur == ctx->device) return AD_OK;
    CUDA_TRY(cudaSetDevice(ctx->device));
    return AD_OK;
}

int32_t report_device_err(int32_t h) {
    return fail(AD_ERR_INVALID_ARG, "a previous kernel reported %s%s%s%s",
                (h & ERR_BAD_LIGAND) ? "[pose_ligand id out of range] " : "",
                (h & ERR_FOOTPRINT) ? "[ligand footprint larger than the launch's] " : "",
                (h & ERR_MIXED_CTA) ? "[pose_ligand not uniform within a CTA group] " : "",
                (h & ERR_STRIDE) ? "[geno_stride < 6 + n_tors of a pose's ligand]" : "");
}

// Surfaces device-side argument errors recorded by earlier kernels without
// blocking: the error word of the last completed read-back (see read_back_err).
// The word is sticky on the device until reported, then cleared in stream order.
int32_t check_device_err(ad_context* ctx, cudaStream_t st) {
    if (!ctx->err_pending) return AD_OK;
    const cudaError_t q = cudaEventQuery(ctx->err_ev);
    if (q == cudaErrorNotReady) return AD_OK;
    if (q != cudaSuccess) return fail(AD_ERR_CUDA, "error read-back: %s", cudaGetErrorString(q));
    ctx->err_pending = false;
    if (*reinterpret_cast<volatile int32_t*>(ctx->h_err) == 0) return AD_OK;
    // an error was flagged: the complete bits from the device word (rare path)
    int32_t h = 0;
    CUDA_TRY(cudaMemcpy(&h, ctx->d_err, sizeof(int32_t), cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemset(ctx->d_err, 0, sizeof(int32_t)));
    *reinterpret_cast<volatile int32_t*>(ctx->h_err) = 0;
    return report_device_err(h ? h : ERR_FOOTPRINT);
}

// Mark this call's launches for the error check of a later call (an event only).
int32_t read_back_err(ad_context* ctx, cudaStream_t st) {
    CUDA_TRY(cudaEventRecord(ctx->err_ev, st));
    ctx->err_pending = true;
    return AD_OK;
}

// Raise a kernel's dynamic shared-memory limit to the device maximum, once.
int32_t opt_in_smem(ad_context* ctx, const void* k) {
    std::lock_guard<std::mutex> lock(ctx->launch_mu);
    if (std::find(ctx->smem_opted.begin(), ctx->smem_opted.end(), k) != ctx->smem_opted.end()) return AD_OK;
    cudaFuncAttributes fa;
    CUDA_TRY(cudaFuncGetAttributes(&fa, k));  // the dynamic limit excludes the kernel's static shared memory
    CUDA_TRY(cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                  ctx->max_smem_optin - (int)fa.sharedSizeBytes));
    ctx->smem_opted.push_back(k);
    return AD_OK;
}

// Resident CTAs per SM of kernel k at (threads, smem), cached.
int32_t occupancy(ad_context* ctx, const void* k, int threads, size_t smem, int* blocks) {
    {
        std::lock_guard<std::mutex> lock(ctx->launch_mu);
        for (const auto& e : ctx->occ)
            if (e[0] == (long long)(uintptr_t)k && e[1] == threads && e[2] == (long long)smem) {
                *blocks = (int)e[3];
                return AD_OK;
            }
    }
    if (int32_t rc = opt_in_smem(ctx, k)) return rc;
    CUDA_TRY(cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, k, threads, smem));
    std::lock_guard<std::mutex> lock(ctx->launch_mu);
    ctx->occ.push_back({(long long)(uintptr_t)k, threads, (long long)smem, *blocks});
    return AD_OK;
}

// Device table of ligands: entry `only` alone when it fits the allocated table
// (uploads of a large screen stay O(1) each), else the whole table.
int32_t sync_ligtab(ad_context* ctx, int only = -1) {
    const int n = (int)ctx->ligs.size();
    if (only >= 0 && only < ctx->ligtab_cap) {
        const LigSlot& L = ctx->ligs[only];
        const LigDev e{L.live ? L.d_blob : nullptr, L.blob_bytes, L.scratch_bytes, L.scratch_simt, L.base_bytes,
                       L.live ? L.d_base : nullptr};
        CUDA_TRY(cudaMemcpy(ctx->d_ligtab + only, &e, sizeof(LigDev), cudaMemcpyHostToDevice));
        return AD_OK;
    }
    if (n > ctx->ligtab_cap) {
        int cap = std::max(64, ctx->ligtab_cap * 2);
        while (cap < n) cap *= 2;
        LigDev* d = nullptr;
        CUDA_TRY(cudaMalloc(&d, sizeof(LigDev) * cap));
        if (ctx->d_ligtab) cudaFree(ctx->d_ligtab);
        ctx->d_ligtab = d;
        ctx->ligtab_cap = cap;
    }
    std::vector<LigDev> h(n);
    for (int i = 0; i < n; ++i)
        h[i] = LigDev{ctx->ligs[i].live ? ctx->ligs[i].d_blob : nullptr, ctx->ligs[i].blob_bytes,
                      ctx->ligs[i].scratch_bytes, ctx->ligs[i].scratch_simt, ctx->ligs[i].base_bytes,
                      ctx->ligs[i].live ? ctx->ligs[i].d_base : nullptr};
    if (n) CUDA_TRY(cudaMemcpy(ctx->d_ligtab, h.data(), sizeof(LigDev) * n, cudaMemcpyHostToDevice));
    return AD_OK;
}

// ---------------------------------------------------------------- blob build
struct BlobBuilder {
    std::vector<unsigned char> buf;
    int32_t put(const void* src, size_t bytes) {
        const int32_t off = (int32_t)buf.size();
        buf.resize(align16(off + (int32_t)bytes), 0);
        if (bytes) memcpy(buf.data() + off, src, bytes);
        return off;
    }
};

struct Schedule {
    int rounds = 0, slots = 1;
    std::vector<uint32_t> rec;  // [rounds*32]
    std::vector<float> dsv;     // scatter: [rounds*64][2] (dsv, cqq); owner / hybrid: [entries] dsv
};

// Swap the roles of i and j in a schedule record (the pair term is symmetric;
// the type-pair index keeps the caller's (i, j) order).
uint32_t swap_ij(uint32_t r) {
    const uint32_t i = r & 0xff, j = (r >> 8) & 0xff, si = (r >> 16) & 0xf, sj = (r >> 20) & 0xf;
    return j | (i << 8) | (sj << 16) | (si << 20) | (r & 0xff000000u);
}

// row stride (float4) of the gradient slots (a multiple of 8, ad_internal.h)
int npad_of(int n_atoms) { return (n_atoms + 7) & ~7; }

// Shared-memory wavefronts of one group of 8 consecutive schedule entries (a
// quarter-warp: the unit in which a 128-bit LDS/STS is serviced, confirmed by ncu
// per-line wavefront counts on configs 2 and 3): for each of the four 128-bit
// accesses of the pair loop (X_i, X_j and the two gradient targets slot * npad +
// atom) the largest number of distinct 16-byte addresses sharing a bank group
// (address / 16 mod 8).  1 per access = conflict free.
int group_cost(const std::pair<int, uint32_t>* e, int npad) {
    int cost = 0;
    for (int acc = 0; acc < 4; ++acc) {
        int addr[8], n = 0;
        for (int k = 0; k < 8; ++k) {
            const uint32_t r = e[k].second;
            const int i = r & 0xff, j = (r >> 8) & 0xff, si = (r >> 16) & 0xf, sj = (r >> 20) & 0xf;
            const int a = acc == 0 ? i : acc == 1 ? j : acc == 2 ? si * npad + i : sj * npad + j;
            bool seen = false;
            for (int t = 0; t < n; ++t) seen |= addr[t] == a;
            if (!seen) addr[n++] = a;
        }
        int per[8] = {0, 0, 0, 0, 0, 0, 0, 0}, mx = 1;
        for (int t = 0; t < n; ++t) mx = std::max(mx, ++per[addr[t] & 7]);
        cost += mx;
    }
    return cost;
}

// Local search over the placement of one step's 64 entries under group_cost:
// swap two entries of different groups, or flip an entry's i/j orientation, when
// that does not raise the cost (deterministic xorshift stream; the set of pairs
// and their gradient slots is unchanged).
void refine_step(std::vector<std::pair<int, uint32_t>>& out, int npad, int iters) {
    uint64_t st = 0x2545F4914F6CDD1Dull;
    auto rnd = [&]() { st ^= st << 13; st ^= st >> 7; st ^= st << 17; return st; };
    int cost[8], cur = 0;
    for (int g = 0; g < 8; ++g) cur += cost[g] = group_cost(&out[g * 8], npad);
    for (int it = 0; it < iters && cur > 32; ++it) {  // 32 = conflict free
        const int a = (int)(rnd() % 64), b = (int)(rnd() % 64);
        const int ga = a / 8, gb = b / 8;
        const bool flip = (rnd() & 3) == 0;
        const auto sa = out[a], sb = out[b];
        if (flip) {
            if (out[a].first < 0) continue;
            out[a].second = swap_ij(out[a].second);
        } else {
            if (ga == gb) continue;
            std::swap(out[a], out[b]);
        }
        const int ca = group_cost(&out[ga * 8], npad);
        const int cb = flip ? 0 : group_cost(&out[gb * 8], npad);
        const int before = cost[ga] + (flip ? 0 : cost[gb]);
        const int after = ca + (flip ? 0 : cb);
        if (after <= before) {
            cost[ga] = ca;
            if (!flip) cost[gb] = cb;
            cur += after - before;
        } else {
            out[a] = sa;
            out[b] = sb;
        }
    }
}

// Place the (<= 64) pairs of one step into 8 groups of 8 consecutive entries
// (= the quarter-warps of the two sub-steps, the unit in which a 128-bit shared
// load/store is serviced).  Within a group the first atoms should have distinct
// residues mod 8 and so should the second atoms: then every LDS.128/STS.128 of
// the pair loop (X_i, X_j, both gradient read-modify-writes, whose addresses are
// slot*npad + atom with npad % 8 == 0) is bank-conflict free.  Greedy, with the
// i/j orientation as a free choice; leftovers fill empty places (then conflicts
// are allowed).  Returns 64 entries, first == -1 marks an empty place.
std::vector<std::pair<int, uint32_t>> arrange_greedy(const std::vector<std::pair<int, uint32_t>>& pool, int n_atoms,
                                                   int K) {
    std::vector<std::pair<int, uint32_t>> out(kPairsPerStep, {-1, 0u});
    std::vector<char> taken(pool.size(), 0);
    int left = (int)pool.size();
    const int groups = kPairsPerStep / 8;
    // spread the load: about ceil(n/8) entries per group
    const int per = (left + groups - 1) / groups;
    for (int g = 0; g < groups && left; ++g) {
        unsigned usedA = 0, usedB = 0;
        int n = 0;
        for (size_t e = 0; e < pool.size() && n < per; ++e) {
            if (taken[e]) continue;
            uint32_t r = pool[e].second;
            unsigned a = r & 7u, b = (r >> 8) & 7u;
            if ((usedA >> a & 1u) || (usedB >> b & 1u)) {
                if ((usedA >> b & 1u) || (usedB >> a & 1u)) continue;
                r = swap_ij(r);
                std::swap(a, b);
            }
            usedA |= 1u << a;
            usedB |= 1u << b;
            out[g * 8 + n] = {pool[e].first, r};
            taken[e] = 1;
            ++n;
            --left;
        }
    }
    for (size_t e = 0, slot = 0; e < pool.size(); ++e) {  // leftovers: any empty place
        if (taken[e]) continue;
        while (out[slot].first >= 0) ++slot;
        out[slot] = pool[e];
    }
    // empty places still issue their loads: point them (i == j == d marks an
    // empty place) at an atom whose residue is unused in the group
    for (int g = 0; g < groups; ++g) {
        unsigned used = 0;
        for (int k = 0; k < 8; ++k)
            if (out[g * 8 + k].first >= 0) used |= (1u << (out[g * 8 + k].second & 7u)) | (1u << ((out[g * 8 + k].second >> 8) & 7u));
        for (int k = 0; k < 8; ++k) {
            if (out[g * 8 + k].first >= 0) continue;
            unsigned d = 0;
            while (d < 8 && d < (unsigned)n_atoms && (used >> d & 1u)) ++d;
            if (d >= 8 || d >= (unsigned)n_atoms) d = 0;
            used |= 1u << d;
            out[g * 8 + k].second = d | (d << 8) | ((uint32_t)K << 16) | ((uint32_t)K << 20);  // spare row K
        }
    }
    return out;
}

// Bank-conflict-minimal placement of one step.  Residue = storage row mod 8 =
// the bank group of every 128-bit access of an atom (X rows and gradient rows
// slot * npad + row, npad % 8 == 0).  A group of 8 entries is conflict free iff
// its 8 i-residues are distinct and its 8 j-residues are distinct, i.e. the group
// is a perfect matching of the bipartite residue multigraph (i-res -> j-res).
//   (1) orient every pair (the pair term is symmetric) so that each residue is an
//       i-end and a j-end about equally often: Euler orientation (odd-degree
//       residues joined to a virtual vertex, edges oriented along closed trails
//       -> |out - in| <= 1 per residue);
//   (2) residues that are still an i-end (j-end) more than 8 times set edges
//       aside (they must share a group with an equal residue: one conflict each);
//   (3) fill every residue up to out = in = 8 with empty places, which may join
//       any two residues (they target the spare row K on both sides and are
//       masked by that slot);
//   (4) peel the 8-regular bipartite multigraph into 8 perfect matchings (Kuhn's
//       augmenting paths; a regular bipartite multigraph always has one, Hall)
//       = the 8 groups;
//   (5) every set-aside edge replaces an empty place, preferring one whose
//       j-residue (i-residue) it matches, so it adds one conflict, not two.
// With at most 16 pair ends per residue in the step (schedule_pairs' cap) and a
// balanced orientation nothing is set aside and the step is conflict free.
bool arrange_matching(const std::vector<std::pair<int, uint32_t>>& pool, int n_atoms, int K,
                      std::vector<std::pair<int, uint32_t>>& out) {
    if (n_atoms < 8 || pool.size() > (size_t)kPairsPerStep) return false;
    const int E = (int)pool.size();
    // (1) orientation: edges between residues, vertex 8 = virtual
    std::vector<int> au(E), av(E);
    int deg[9] = {0};
    for (int e = 0; e < E; ++e) {
        au[e] = pool[e].second & 7u;
        av[e] = (pool[e].second >> 8) & 7u;
        deg[au[e]]++;
        deg[av[e]]++;
    }
    for (int r = 0; r < 8; ++r)
        if (deg[r] & 1) { au.push_back(r); av.push_back(8); }
    const int EA = (int)au.size();
    std::vector<std::vector<int>> inc(9);
    for (int e = 0; e < EA; ++e) { inc[au[e]].push_back(e); inc[av[e]].push_back(e); }
    std::vector<char> used(EA, 0), fwd(EA, 1);  // fwd: traversed au -> av
    std::vector<size_t> ptr(9, 0);
    for (int start = 0; start < 9; ++start) {
        for (;;) {  // closed trails from `start` while it has unused edges
            while (ptr[start] < inc[start].size() && used[inc[start][ptr[start]]]) ptr[start]++;
            if (ptr[start] == inc[start].size()) break;
            int v = start;
            do {
                while (used[inc[v][ptr[v]]]) ptr[v]++;  // every vertex has even unused degree
                const int e = inc[v][ptr[v]];
                used[e] = 1;
                fwd[e] = au[e] == v;
                v = fwd[e] ? av[e] : au[e];
            } while (v != start);
        }
    }
    int outd[8] = {0}, ind[8] = {0};
    std::vector<uint32_t> rec;
    std::vector<int> ids;
    std::vector<std::pair<int, uint32_t>> aside;
    for (int e = 0; e < E; ++e) {
        const uint32_t r = fwd[e] ? pool[e].second : swap_ij(pool[e].second);
        const int ro = r & 7u, ri = (r >> 8) & 7u;
        // (2) over-full residues set the edge aside
        if (outd[ro] == 8 || ind[ri] == 8) {
            aside.push_back({pool[e].first, r});
            continue;
        }
        outd[ro]++;
        ind[ri]++;
        rec.push_back(r);
        ids.push_back(pool[e].first);
    }
    // (3) empty places: i-residue with an out deficit -> j-residue with an in deficit;
    // rows 0..7 hold real atoms (balance_slots), their X rows are real positions
    int ro = 0, ri = 0;
    while ((int)rec.size() < kPairsPerStep) {
        while (outd[ro] == 8) ++ro;
        while (ind[ri] == 8) ++ri;
        outd[ro]++;
        ind[ri]++;
        rec.push_back((uint32_t)ro | ((uint32_t)ri << 8) | ((uint32_t)K << 16) | ((uint32_t)K << 20));
        ids.push_back(-1);
    }
    // (4) peel 8 perfect matchings
    std::vector<int> bucket[8][8];
    for (int e = 0; e < kPairsPerStep; ++e) bucket[rec[e] & 7u][(rec[e] >> 8) & 7u].push_back(e);
    out.assign(kPairsPerStep, {-1, 0u});
    struct Aug {
        std::vector<int> (*b)[8];
        int* mr;
        bool* sn;
        bool run(int x) {
            for (int v = 0; v < 8; ++v) {
                if (b[x][v].empty() || sn[v]) continue;
                sn[v] = true;
                if (mr[v] < 0 || run(mr[v])) { mr[v] = x; return true; }
            }
            return false;
        }
    };
    for (int g = 0; g < 8; ++g) {
        int match_r[8];  // right vertex -> left vertex
        for (int v = 0; v < 8; ++v) match_r[v] = -1;
        for (int u = 0; u < 8; ++u) {
            bool seen[8] = {false, false, false, false, false, false, false, false};
            Aug aug{bucket, match_r, seen};
            if (!aug.run(u)) return false;  // cannot happen for a regular multigraph
        }
        for (int v = 0; v < 8; ++v) {
            const int u = match_r[v];
            const int e = bucket[u][v].back();
            bucket[u][v].pop_back();
            out[g * 8 + u] = {ids[e], rec[e]};
        }
    }
    // (5) set-aside edges replace empty places (one conflict when a residue matches)
    for (const auto& x : aside) {
        const int xo = x.second & 7u, xi = (x.second >> 8) & 7u;
        int best = -1, bscore = -1;
        for (int q = 0; q < kPairsPerStep; ++q) {
            if (out[q].first >= 0) continue;
            const int sc = ((int)(out[q].second & 7u) == xo) + ((int)((out[q].second >> 8) & 7u) == xi);
            if (sc > bscore) { bscore = sc; best = q; }
        }
        if (best < 0) return false;  // cannot happen: E <= 64
        out[best] = x;
    }
    return true;
}

std::vector<std::pair<int, uint32_t>> arrange_step(const std::vector<std::pair<int, uint32_t>>& pool, int n_atoms,
                                                   int K, int refine_iters) {
    // two candidates, the lower modelled cost wins: the matching construction (exact
    // when the step's residues allow it) and the greedy grouping; both polished by
    // the local search unless already conflict free
    const int npad = npad_of(n_atoms);
    auto total = [&](const std::vector<std::pair<int, uint32_t>>& o) {
        int c = 0;
        for (int g = 0; g < 8; ++g) c += group_cost(&o[g * 8], npad);
        return c;
    };
    std::vector<std::pair<int, uint32_t>> m;
    int cm = 1 << 30;
    if (!getenv("AD_NO_MATCHING") && arrange_matching(pool, n_atoms, K, m)) {
        cm = total(m);
        if (cm > 32) {
            refine_step(m, npad, refine_iters);
            cm = total(m);
        }
        if (cm == 32 || getenv("AD_MATCHING_ONLY")) return m;  // 4 accesses x 8 groups x 1 wavefront
    }
    std::vector<std::pair<int, uint32_t>> g = arrange_greedy(pool, n_atoms, K);
    refine_step(g, npad, refine_iters);
    return total(g) < cm ? g : m;
}

// Storage row of every atom (INTRA_SCATTER): the row picks the bank group
// (row mod 8) of the atom's X row and gradient rows.  A step can only be placed
// conflict free (arrange_matching) when no bank group carries more than 16 pair
// ends in it, so the bank groups should carry equal numbers of pair ends.  The
// per-atom phases (pose, gradient sums) access atoms a = lane + 32 m, i.e. every
// aligned octet of atoms within one quarter-warp: rows are therefore only
// permuted WITHIN each octet (rows 8m .. 8m+7 stay the octet's, so those
// accesses stay conflict free), heaviest atom of the octet to the least loaded
// bank group so far.
std::vector<int> balance_slots(int n_atoms, const std::vector<int>& pi, const std::vector<int>& pj) {
    std::vector<int> slot(n_atoms);
    for (int a = 0; a < n_atoms; ++a) slot[a] = a;
    if (n_atoms < 8 || getenv("AD_NO_BALANCE")) return slot;
    std::vector<int> ends(n_atoms, 0);
    for (size_t q = 0; q < pi.size(); ++q) {
        ends[pi[q]]++;
        ends[pj[q]]++;
    }
    long load[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (int base = 0; base < n_atoms; base += 8) {
        const int n = std::min(8, n_atoms - base);
        int ord[8];
        for (int k = 0; k < n; ++k) ord[k] = base + k;
        std::stable_sort(ord, ord + n, [&](int x, int y) { return ends[x] > ends[y]; });
        bool taken[8] = {false, false, false, false, false, false, false, false};
        for (int k = 0; k < n; ++k) {
            int best = -1;
            for (int r = 0; r < 8; ++r)
                if (!taken[r] && (best < 0 || load[r] < load[best])) best = r;
            taken[best] = true;
            slot[ord[k]] = base + best;
            load[best] += ends[ord[k]];
        }
    }
    return slot;
}

// Swap pairs between steps (or move them into free places) until no bank group
// (row mod 8) carries more than 16 pair ends in any step, keeping every atom at
// most K times per step: arrange_matching can then place every step conflict
// free.  Deterministic (fixed xorshift stream); returns the remaining overload.
int rebalance_steps(std::vector<std::vector<int>>& steps, const std::vector<int>& pi, const std::vector<int>& pj,
                    int n_idx, int K, long iters) {
    const int R = (int)steps.size();
    if (R < 2) return 0;
    const int cap = 2 * kPairsPerStep / 8;
    std::vector<std::vector<uint8_t>> cnt(R, std::vector<uint8_t>(n_idx, 0));
    std::vector<std::array<int, 8>> deg(R);
    auto over = [&](const std::array<int, 8>& d) {
        int o = 0;
        for (int r = 0; r < 8; ++r) o += std::max(0, d[r] - cap);
        return o;
    };
    int total = 0;
    for (int a = 0; a < R; ++a) {
        deg[a].fill(0);
        for (int q : steps[a]) {
            cnt[a][pi[q]]++;
            cnt[a][pj[q]]++;
            deg[a][pi[q] & 7]++;
            deg[a][pj[q] & 7]++;
        }
        total += over(deg[a]);
    }
    // lower bound: a bank group with more than cap * R ends overall stays overloaded
    // however the pairs are spread (stop there instead of spending all iterations)
    int bound = 0;
    {
        int g_all[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        for (int a = 0; a < R; ++a)
            for (int r = 0; r < 8; ++r) g_all[r] += deg[a][r];
        for (int r = 0; r < 8; ++r) bound += std::max(0, g_all[r] - cap * R);
    }
    uint64_t st = 0xD1B54A32D192ED03ull;
    auto rnd = [&]() { st ^= st << 13; st ^= st >> 7; st ^= st << 17; return st; };
    for (long it = 0; it < iters && total > bound; ++it) {
        const int A = (int)(rnd() % R), B = (int)(rnd() % R);
        if (A == B || steps[A].empty()) continue;
        if (over(deg[A]) == 0 && over(deg[B]) == 0) continue;
        const int ia = (int)(rnd() % steps[A].size());
        const int p = steps[A][ia];
        // q = a pair of B, or (-1) a free place of B
        const int nb = (int)steps[B].size() + (steps[B].size() < (size_t)kPairsPerStep ? 1 : 0);
        const int ib = (int)(rnd() % nb);
        const int q = ib < (int)steps[B].size() ? steps[B][ib] : -1;
        // K limits after the exchange
        auto ok_into = [&](int S, int in, int outp) {
            const int a = pi[in], b = pj[in];
            int ca = cnt[S][a] + 1, cb = cnt[S][b] + 1;
            if (outp >= 0) {
                if (pi[outp] == a || pj[outp] == a) ca--;
                if (pi[outp] == b || pj[outp] == b) cb--;
            }
            return ca <= K && cb <= K;
        };
        if (!ok_into(B, p, q) || (q >= 0 && !ok_into(A, q, p))) continue;
        std::array<int, 8> dA = deg[A], dB = deg[B];
        dA[pi[p] & 7]--; dA[pj[p] & 7]--; dB[pi[p] & 7]++; dB[pj[p] & 7]++;
        if (q >= 0) { dB[pi[q] & 7]--; dB[pj[q] & 7]--; dA[pi[q] & 7]++; dA[pj[q] & 7]++; }
        const int before = over(deg[A]) + over(deg[B]), after = over(dA) + over(dB);
        if (after > before) continue;
        // apply
        cnt[A][pi[p]]--; cnt[A][pj[p]]--; cnt[B][pi[p]]++; cnt[B][pj[p]]++;
        if (q >= 0) {
            cnt[B][pi[q]]--; cnt[B][pj[q]]--; cnt[A][pi[q]]++; cnt[A][pj[q]]++;
            steps[A][ia] = q;
            steps[B][ib] = p;
        } else {
            steps[A][ia] = steps[A].back();
            steps[A].pop_back();
            steps[B].push_back(p);
        }
        deg[A] = dA;
        deg[B] = dB;
        total += after - before;
    }
    return total;
}

// pdsv / pcq: per pair desolvation prefactor and coeff_el q_i q_j; the schedule
// stores them interleaved (float2 per entry; empty places (0, 0))
// effort (ad_set_schedule_effort): 2 = full placement search (the default; ~1-500 ms
// of host time per ligand), 1 = a tenth of the local-search iterations, 0 = no
// cross-step rebalancing and no local search (matching / greedy construction only).
Schedule schedule_pairs(int n_atoms, const std::vector<int>& pi, const std::vector<int>& pj,
                        const std::vector<int>& ptp, const std::vector<float>& pdsv, const std::vector<float>& pcq,
                        int effort = 2) {
    static const int refine_env = getenv("AD_REFINE_ITERS") ? atoi(getenv("AD_REFINE_ITERS")) : -1;
    const int refine_iters = refine_env >= 0 ? refine_env : effort >= 2 ? 20000 : effort == 1 ? 2000 : 0;
    const long rebalance_per_step = effort >= 2 ? 200000L : effort == 1 ? 20000L : 0L;
    const int P = (int)pi.size();
    const int target = (P + kPairsPerStep - 1) / kPairsPerStep;
    Schedule best;
    best.rounds = 1 << 30;
    std::vector<int> perm(P);
    for (int q = 0; q < P; ++q) perm[q] = q;
    uint64_t st = 0x9E3779B97F4A7C15ull;
    for (int q = P - 1; q > 0; --q) {  // Fisher-Yates with a fixed xorshift stream
        st ^= st << 13; st ^= st >> 7; st ^= st << 17;
        std::swap(perm[q], perm[(int)(st % (uint64_t)(q + 1))]);
    }
    const int kmax = std::min(8, std::max(2, 256 / std::max(n_atoms, 1)));
    const int n_idx = npad_of(n_atoms);  // atom indices are storage slots (< npad)
    std::vector<std::vector<std::pair<int, uint32_t>>> best_rounds;
    // capped: at most 16 pair ends per bank group and step (arrange_matching's
    // precondition); uncapped as a fallback when the cap costs a step
    for (int capped = 1; capped >= 0; --capped)
    for (int K = 1; K <= kmax; ++K) {
        if (!capped && best.rounds <= target) break;
        std::vector<int> rem = perm;
        std::vector<std::vector<std::pair<int, uint32_t>>> rounds;
        std::vector<int> cnt(n_idx);
        const int rcap = (capped && n_atoms >= 8) ? 2 * kPairsPerStep / 8 : 1 << 30;
        while (!rem.empty()) {
            std::fill(cnt.begin(), cnt.end(), 0);
            int rc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
            std::vector<std::pair<int, uint32_t>> rnd;
            std::vector<int> rest;
            for (int q : rem) {
                const int i = pi[q], j = pj[q];
                const int need_i = 1 + ((i & 7) == (j & 7)), need_j = need_i;
                if ((int)rnd.size() < kPairsPerStep && cnt[i] < K && cnt[j] < K && rc[i & 7] + need_i <= rcap &&
                    rc[j & 7] + need_j <= rcap) {
                    rc[i & 7]++;
                    rc[j & 7]++;
                    const uint32_t r = (uint32_t)i | ((uint32_t)j << 8) | ((uint32_t)cnt[i] << 16) |
                                       ((uint32_t)cnt[j] << 20) | ((uint32_t)ptp[q] << 24);
                    cnt[i]++;
                    cnt[j]++;
                    rnd.push_back({q, r});
                } else {
                    rest.push_back(q);
                }
            }
            rounds.push_back(std::move(rnd));
            rem.swap(rest);
        }
        const int R = (int)rounds.size();
        if (getenv("AD_DEBUG_SCHEDULE")) fprintf(stderr, "[libad] schedule capped=%d K=%d rounds=%d (target %d)\n", capped, K, R, target);
        if (R < best.rounds) {
            best.rounds = R;
            best.slots = K;
            best_rounds = std::move(rounds);
        }
        if (R <= target) break;
    }
    (void)target;
    if (n_atoms >= 8 && rebalance_per_step > 0 && !getenv("AD_NO_REBALANCE")) {
        // cross-step rebalancing, then slots re-assigned by occurrence order
        std::vector<std::vector<int>> ids(best_rounds.size());
        for (size_t r = 0; r < best_rounds.size(); ++r)
            for (const auto& e : best_rounds[r]) ids[r].push_back(e.first);
        const int left = rebalance_steps(ids, pi, pj, n_idx, best.slots, rebalance_per_step * (long)ids.size());
        if (getenv("AD_DEBUG_SCHEDULE")) fprintf(stderr, "[libad] rebalance: overload left %d\n", left);
        std::vector<int> cnt(n_idx);
        for (size_t r = 0; r < ids.size(); ++r) {
            std::fill(cnt.begin(), cnt.end(), 0);
            best_rounds[r].clear();
            for (int q : ids[r]) {
                const int i = pi[q], j = pj[q];
                best_rounds[r].push_back({q, (uint32_t)i | ((uint32_t)j << 8) | ((uint32_t)cnt[i] << 16) |
                                                 ((uint32_t)cnt[j] << 20) | ((uint32_t)ptp[q] << 24)});
                cnt[i]++;
                cnt[j]++;
            }
        }
    }
    // entry l of step r goes to lane l % 32, sub-step l / 32: index (2r + l/32)*32 + l%32 = 64r + l
    best.rec.assign((size_t)best_rounds.size() * kPairsPerStep, 0u);
    best.dsv.assign((size_t)best_rounds.size() * kPairsPerStep * 2, 0.f);
    // steps are arranged independently (deterministic per step): spread them over
    // the host's cores
    std::atomic<size_t> next{0};
    auto worker = [&]() {
        for (size_t r; (r = next.fetch_add(1)) < best_rounds.size();) {
            const std::vector<std::pair<int, uint32_t>> lay = arrange_step(best_rounds[r], n_atoms, best.slots, refine_iters);
            for (int l = 0; l < kPairsPerStep; ++l) {
                best.rec[r * kPairsPerStep + l] = lay[l].second;
                best.dsv[2 * (r * kPairsPerStep + l)] = lay[l].first < 0 ? 0.f : pdsv[lay[l].first];
                best.dsv[2 * (r * kPairsPerStep + l) + 1] = lay[l].first < 0 ? 0.f : pcq[lay[l].first];
            }
        }
    };
    const size_t n_thr = std::min<size_t>(best_rounds.size(), std::max(1u, std::thread::hardware_concurrency()));
    std::vector<std::thread> pool;
    for (size_t t = 1; t < n_thr; ++t) pool.emplace_back(worker);
    worker();
    for (auto& t : pool) t.join();
    if (P == 0) {
        best.rounds = 0;
        best.slots = 1;
    }
    return best;
}

// ---------------------------------------------------------------------------
// Cherry schedule: the shared-memory mode of INTRA_SCATTER (kernel side:
// intra_cherry).  Rows are storage rows (< npad).
//   (1) cherries: every pair becomes an end of a cherry (c; e0, e1) = the pairs
//       (c, e0), (c, e1).  Atoms are visited by descending degree; each pairs up
//       its remaining pairs two by two as cherries centred on itself, holding one
//       back (towards an unvisited atom) when the count is odd.  A connected pair
//       graph with an even pair count decomposes completely into cherries; what is
//       left over becomes a single (one empty end).  High-degree atoms become
//       centres, which evens out the per-atom target load (a centre is ONE
//       gradient target for two pairs).
//   (2) steps: greedy first-fit of the cherries into steps of 32 lanes with at
//       most K targets per atom and step (slots 0..K-1): the smallest K reaching
//       the fewest steps.  Capped at 4 centres and 8 ends per bank group and step
//       (a precondition of a conflict-free placement) unless the cap costs a step.
//   (3) placement: local search over the lane positions (quarter-warps of 8
//       lanes; swaps within and across steps that keep every step within K
//       targets per atom) and the end order of every cherry, minimising the
//       shared-memory wavefronts: sum over quarter-warps and the three 128-bit
//       accesses (centre, end 0, end 1) of the largest number of lanes sharing a
//       bank group (row % 8; X rows and gradient rows of an atom share it, npad %
//       8 == 0).  Config 2 reaches 13.5 wavefronts per step-quarter set (ideal 12).
struct CherryLane {
    int c = -1, e[2] = {-1, -1}, p[2] = {-1, -1};  // rows; pair ids (-1: empty end / lane)
    int kc = -1, ke[2] = {-1, -1};                  // slots of the targets
};
struct CherrySchedule {
    int steps = 0, slots = 1;
    std::vector<CherryLane> lane;  // [steps * 32]
};

std::vector<CherryLane> make_cherries(int n_idx, const std::vector<int>& pi, const std::vector<int>& pj) {
    const int P = (int)pi.size();
    std::vector<std::vector<int>> inc(n_idx);
    for (int q = 0; q < P; ++q) {
        inc[pi[q]].push_back(q);
        inc[pj[q]].push_back(q);
    }
    std::vector<int> order(n_idx);
    for (int a = 0; a < n_idx; ++a) order[a] = a;
    std::stable_sort(order.begin(), order.end(), [&](int x, int y) { return inc[x].size() > inc[y].size(); });
    std::vector<char> used(P, 0), visited(n_idx, 0);
    auto other = [&](int q, int a) { return pi[q] == a ? pj[q] : pi[q]; };
    std::vector<CherryLane> out;
    for (int a : order) {
        std::vector<int> rem;
        for (int q : inc[a])
            if (!used[q]) rem.push_back(q);
        visited[a] = 1;
        if (rem.size() % 2)  // hold back one pair towards an unvisited atom: it pairs up there
            for (size_t k = 0; k < rem.size(); ++k)
                if (!visited[other(rem[k], a)]) {
                    rem.erase(rem.begin() + (long)k);
                    break;
                }
        // two pairs of one cherry must end on different atoms (duplicate pairs)
        while (rem.size() >= 2) {
            const int q0 = rem.back();
            rem.pop_back();
            size_t k = rem.size();
            while (k > 0 && other(rem[k - 1], a) == other(q0, a)) --k;
            if (k == 0) break;  // q0 stays unused: a single below
            const int q1 = rem[k - 1];
            rem.erase(rem.begin() + (long)(k - 1));
            CherryLane L;
            L.c = a;
            L.e[0] = other(q0, a);
            L.e[1] = other(q1, a);
            L.p[0] = q0;
            L.p[1] = q1;
            used[q0] = used[q1] = 1;
            out.push_back(L);
        }
    }
    for (int q = 0; q < P; ++q)
        if (!used[q]) {
            CherryLane L;
            L.c = pi[q];
            L.e[0] = pj[q];
            L.p[0] = q;
            out.push_back(L);
        }
    return out;
}

// wavefronts of one quarter-warp (8 lanes): sum over the three accesses of the
// largest number of lanes in one bank group; empty ends / lanes do not count
// (they get a free bank group later)
int cherry_quarter_cost(const CherryLane* const* q, const uint8_t* flip) {
    int cost = 0;
    for (int acc = 0; acc < 3; ++acc) {
        int cnt[8] = {0, 0, 0, 0, 0, 0, 0, 0}, mx = 0;
        for (int l = 0; l < 8; ++l) {
            if (!q[l] || q[l]->c < 0) continue;
            const int row = acc == 0 ? q[l]->c : q[l]->e[(acc - 1) ^ flip[l]];
            if (row < 0) continue;
            mx = std::max(mx, ++cnt[row & 7]);
        }
        cost += mx;
    }
    return cost;
}

// max_steps: a schedule with more steps is not placed (steps is still reported);
// max_K: the most gradient slots the records can address (8-bit rows, cherry_rows_fit)
CherrySchedule schedule_cherries(int n_idx, const std::vector<int>& pi, const std::vector<int>& pj, int effort,
                                 int max_steps = 1 << 30, int max_K = 8) {
    CherrySchedule S;
    std::vector<CherryLane> ch = make_cherries(n_idx, pi, pj);
    const int n = (int)ch.size();
    if (n == 0) return S;
    {  // deterministic shuffle (first-fit order)
        uint64_t st = 0x2545F4914F6CDD1Dull;
        for (int q = n - 1; q > 0; --q) {
            st ^= st << 13; st ^= st >> 7; st ^= st << 17;
            std::swap(ch[q], ch[(int)(st % (uint64_t)(q + 1))]);
        }
    }
    const int target = (n + 31) / 32;
    std::vector<std::vector<int>> best;
    int bestK = 0;
    for (int capped = 1; capped >= 0; --capped) {
        for (int K = 1; K <= max_K; ++K) {
            if (!best.empty() && (int)best.size() <= target) break;
            std::vector<std::vector<int>> steps;
            std::vector<int> rem(n), cnt(n_idx);
            for (int q = 0; q < n; ++q) rem[q] = q;
            while (!rem.empty()) {
                std::fill(cnt.begin(), cnt.end(), 0);
                int rc[8] = {0, 0, 0, 0, 0, 0, 0, 0}, re[8] = {0, 0, 0, 0, 0, 0, 0, 0};
                std::vector<int> st, rest;
                for (int x : rem) {
                    const CherryLane& L = ch[x];
                    bool ok = st.size() < 32 && cnt[L.c] < K && cnt[L.e[0]] < K && (L.e[1] < 0 || cnt[L.e[1]] < K);
                    if (ok && capped) {
                        int ne[8] = {0, 0, 0, 0, 0, 0, 0, 0};
                        ne[L.e[0] & 7]++;
                        if (L.e[1] >= 0) ne[L.e[1] & 7]++;
                        ok = rc[L.c & 7] < 4;
                        for (int r = 0; r < 8 && ok; ++r) ok = re[r] + ne[r] <= 8;
                    }
                    if (!ok) {
                        rest.push_back(x);
                        continue;
                    }
                    st.push_back(x);
                    cnt[L.c]++;
                    cnt[L.e[0]]++;
                    if (L.e[1] >= 0) cnt[L.e[1]]++;
                    rc[L.c & 7]++;
                    re[L.e[0] & 7]++;
                    if (L.e[1] >= 0) re[L.e[1] & 7]++;
                }
                steps.push_back(std::move(st));
                rem.swap(rest);
            }
            if (best.empty() || steps.size() < best.size()) {
                best = std::move(steps);
                bestK = K;
            }
        }
        if ((int)best.size() <= target) break;
    }
    S.steps = (int)best.size();
    S.slots = bestK;
    if (S.steps > max_steps) return S;
    {   // spread the empty lanes: first-fit leaves them all in the last steps, where their
        // dummy gradient targets cannot all get distinct rows (pack_cherries); move cherries
        // from full steps into deficient ones (within K) until every step holds at least
        // 32 - ceil(empty / steps) cherries
        const int n_empty = S.steps * 32 - n, lo = 32 - (n_empty + S.steps - 1) / S.steps;
        std::vector<int> c2((size_t)S.steps * n_idx, 0);
        for (int st = 0; st < S.steps; ++st)
            for (int x : best[st]) {
                const CherryLane& L = ch[x];
                c2[(size_t)st * n_idx + L.c]++;
                for (int k = 0; k < 2; ++k)
                    if (L.e[k] >= 0) c2[(size_t)st * n_idx + L.e[k]]++;
            }
        auto fits_in = [&](int st, const CherryLane& L) {
            if (c2[(size_t)st * n_idx + L.c] >= bestK) return false;
            for (int k = 0; k < 2; ++k)
                if (L.e[k] >= 0 && c2[(size_t)st * n_idx + L.e[k]] >= bestK) return false;
            return true;
        };
        auto move = [&](int from, size_t idx, int to) {
            const int x = best[from][idx];
            const CherryLane& L = ch[x];
            for (int k = -1; k < 2; ++k) {
                const int a = k < 0 ? L.c : L.e[k];
                if (a < 0) continue;
                c2[(size_t)from * n_idx + a]--;
                c2[(size_t)to * n_idx + a]++;
            }
            best[to].push_back(x);
            best[from].erase(best[from].begin() + (long)idx);
        };
        for (int to = 0; to < S.steps; ++to) {
            for (int from = 0; from < S.steps && (int)best[to].size() < lo; ++from) {
                if (from == to) continue;
                for (size_t i = 0; i < best[from].size() && (int)best[from].size() > lo && (int)best[to].size() < lo;) {
                    if (fits_in(to, ch[best[from][i]])) move(from, i, to); else ++i;
                }
            }
        }
    }
    S.lane.assign((size_t)S.steps * 32, CherryLane{});
    // (3) placement: one local search over all positions (swaps within and across
    // steps that keep every step within K targets per atom, and end flips)
    const int NP = S.steps * 32, K = bestK;
    std::vector<const CherryLane*> pos(NP, nullptr);
    std::vector<uint8_t> flip(NP, 0);
    std::vector<int> cnt((size_t)S.steps * n_idx, 0);
    for (int st = 0; st < S.steps; ++st)
        for (size_t l = 0; l < best[st].size(); ++l) {
            const CherryLane* L = &ch[best[st][l]];
            pos[st * 32 + (int)l] = L;
            cnt[(size_t)st * n_idx + L->c]++;
            for (int k = 0; k < 2; ++k)
                if (L->e[k] >= 0) cnt[(size_t)st * n_idx + L->e[k]]++;
        }
    std::vector<int> qc(NP / 8);
    for (int g = 0; g < NP / 8; ++g) qc[g] = cherry_quarter_cost(&pos[8 * g], &flip[8 * g]);
    auto fits = [&](int st, const CherryLane* in, const CherryLane* out) {  // K after swapping `out` for `in` in step st
        if (!in) return true;
        const int at[3] = {in->c, in->e[0], in->e[1]};
        for (int k = 0; k < 3; ++k) {
            if (at[k] < 0) continue;
            int c = cnt[(size_t)st * n_idx + at[k]] + 1;
            if (out && (out->c == at[k] || out->e[0] == at[k] || out->e[1] == at[k])) --c;
            if (c > K) return false;
        }
        return true;
    };
    auto move_cnt = [&](int st, const CherryLane* L, int d) {
        if (!L) return;
        cnt[(size_t)st * n_idx + L->c] += d;
        for (int k = 0; k < 2; ++k)
            if (L->e[k] >= 0) cnt[(size_t)st * n_idx + L->e[k]] += d;
    };
    // greedy local search (moves that do not add wavefronts), half of the moves
    // targeted at a lane on a conflicting bank group; 400k moves per step at effort 2
    // (config 2: ~0.4 s of host time at upload), a tenth at effort 1; long schedules
    // (global-memory cherries, config 3: 89 steps) get the budget of 48 steps
    static const long imul = getenv("AD_CHERRY_ITERS") ? atol(getenv("AD_CHERRY_ITERS")) : 400000;
    const long iters = (long)(effort >= 2 ? imul : effort == 1 ? imul / 10 : 0) * std::min(S.steps, 48);
    uint64_t rng = 0x9E3779B97F4A7C15ull;
    int total = 0, floor_cost = 0;  // floor: 3 per quarter-warp holding a cherry
    for (int g = 0; g < NP / 8; ++g) total += qc[g];
    for (int st = 0; st < S.steps; ++st) floor_cost += 3 * (((int)best[st].size() + 7) / 8);
    for (long it = 0; it < iters && total > floor_cost; ++it) {
        rng ^= rng << 13; rng ^= rng >> 7; rng ^= rng << 17;
        int a = (int)(rng % (uint64_t)NP);
        const int b = (int)((rng >> 24) % (uint64_t)NP);
        if ((rng >> 40) & 1) {  // targeted: a lane on a bank group that conflicts in its quarter-warp
            const int g = a >> 3;
            if (qc[g] > 3) {
                int best_acc = -1, best_r = -1, mx = 1;
                for (int acc = 0; acc < 3; ++acc) {
                    int c8[8] = {0, 0, 0, 0, 0, 0, 0, 0};
                    for (int l = 8 * g; l < 8 * g + 8; ++l) {
                        if (!pos[l]) continue;
                        const int row = acc == 0 ? pos[l]->c : pos[l]->e[(acc - 1) ^ flip[l]];
                        if (row >= 0 && ++c8[row & 7] > mx) { mx = c8[row & 7]; best_acc = acc; best_r = row & 7; }
                    }
                }
                if (best_acc >= 0) {
                    const int start = (int)((rng >> 48) & 7);
                    for (int k = 0; k < 8; ++k) {
                        const int l = 8 * g + ((start + k) & 7);
                        if (!pos[l]) continue;
                        const int row = best_acc == 0 ? pos[l]->c : pos[l]->e[(best_acc - 1) ^ flip[l]];
                        if (row >= 0 && (row & 7) == best_r) { a = l; break; }
                    }
                }
            }
        }
        const int ga = a >> 3, gb = b >> 3;
        if ((rng >> 50) % 4 == 0) {  // flip the ends of position a
            if (!pos[a]) continue;
            flip[a] ^= 1;
            const int c = cherry_quarter_cost(&pos[8 * ga], &flip[8 * ga]);
            if (c <= qc[ga]) { total += c - qc[ga]; qc[ga] = c; } else flip[a] ^= 1;
            continue;
        }
        if (ga == gb || (!pos[a] && !pos[b])) continue;
        const int sa = a >> 5, sb = b >> 5;
        if (sa != sb && (!fits(sa, pos[b], pos[a]) || !fits(sb, pos[a], pos[b]))) continue;
        std::swap(pos[a], pos[b]);
        std::swap(flip[a], flip[b]);
        // the moved cherries take their best end orientation at the new positions
        int ca = 0, cb = 0;
        const uint8_t fa0 = flip[a], fb0 = flip[b];
        {
            int best_c = 1 << 30;
            uint8_t bfa = fa0, bfb = fb0;
            for (int m = 0; m < 4; ++m) {
                flip[a] = fa0 ^ (uint8_t)(m & 1);
                flip[b] = fb0 ^ (uint8_t)(m >> 1);
                const int x = cherry_quarter_cost(&pos[8 * ga], &flip[8 * ga]);
                const int y = cherry_quarter_cost(&pos[8 * gb], &flip[8 * gb]);
                if (x + y < best_c) { best_c = x + y; ca = x; cb = y; bfa = flip[a]; bfb = flip[b]; }
            }
            flip[a] = bfa;
            flip[b] = bfb;
        }
        if (ca + cb <= qc[ga] + qc[gb]) {
            total += ca + cb - qc[ga] - qc[gb];
            qc[ga] = ca;
            qc[gb] = cb;
            if (sa != sb) {  // pos[a] came from step sb, pos[b] from step sa
                move_cnt(sa, pos[b], -1);
                move_cnt(sa, pos[a], +1);
                move_cnt(sb, pos[a], -1);
                move_cnt(sb, pos[b], +1);
            }
        } else {
            flip[a] = fa0;
            flip[b] = fb0;
            std::swap(pos[a], pos[b]);
            std::swap(flip[a], flip[b]);
        }
    }
    for (int st = 0; st < S.steps; ++st) {
        std::vector<int> c(n_idx, 0);
        for (int l = 0; l < 32; ++l) {
            CherryLane& o = S.lane[(size_t)st * 32 + l];
            const CherryLane* src = pos[st * 32 + l];
            if (!src) continue;
            o = *src;
            if (flip[st * 32 + l]) {
                std::swap(o.e[0], o.e[1]);
                std::swap(o.p[0], o.p[1]);
            }
            o.kc = c[o.c]++;
            for (int k = 0; k < 2; ++k) o.ke[k] = o.e[k] >= 0 ? c[o.e[k]]++ : -1;
        }
    }
    return S;
}

// Records of a cherry schedule (layout: ad_internal.h pka / pkb / pkc, kernel:
// intra_cherry).  Empty ends and lanes get a zero-charge X row and a dummy
// gradient row in the bank group least used by that access in their
// quarter-warp (distinct groups within a lane).  distinct = true: the dummy rows
// of one step are all different (row K * npad + r, r = group + 8 m, the smallest
// free m), so the kernel stores unconditionally and no two lanes of a step touch
// one row; n_spare = the spare rows that takes (a multiple of 8).  distinct =
// false: dummies share the 8 rows K * npad + group and carry "empty" flags (a.y
// bits 24-26) for the predicated loop (PK_PRED).  Row indices are 8-bit: X row
// (< npad + 8) and gradient row k * npad + row (< K * npad + n_spare), both <= 255
// (cherry_rows_fit).
struct CherryRecords {
    std::vector<uint4> a;
    std::vector<float4> b;
    std::vector<float4> c;   // 48-B records (shared-memory cherries): (r0, r0', -cC, -cC')
    std::vector<float2> c2;  // 40-B records (global-memory cherries): (r0, r0')
    int n_spare = 8;
};
bool cherry_rows_fit(int npad, int K) { return npad + 8 <= 256 && K * npad + 8 <= 256; }
int cherry_max_slots(int npad) { return npad + 8 <= 256 ? std::min(8, (256 - 8) / npad) : 0; }

// compact: the 40-B record of the global-memory cherry loop (intra_cherry_gm): each pair's one
// nonzero dispersion coefficient in b, its 12-10 flag in a.x bits 24-25 (config 3: 108.2 ->
// 104.7 ms per LS launch, the loop being L1-bound; bit-identical).  The shared-memory loop keeps
// the 48-B record: its 80-register kernel pays more for the selects than it saves (2.99 -> 3.02 ms).
CherryRecords pack_cherries(const CherrySchedule& S, int npad, const std::vector<int>& ptp,
                            const std::vector<float4>& tp, const std::vector<float>& pdsv, bool distinct,
                            bool compact) {
    CherryRecords R;
    const size_t n = (size_t)S.steps * 32;
    R.a.resize(n);
    R.b.resize(n);
    if (compact) R.c2.resize(n); else R.c.resize(n);
    const int K = S.slots;
    uint64_t step_used[4] = {0, 0, 0, 0};  // dummy rows (0..255) taken in the current step
    for (size_t q0 = 0; q0 < n; q0 += 8) {  // one quarter-warp
        if (q0 % 32 == 0) step_used[0] = step_used[1] = step_used[2] = step_used[3] = 0;
        int cnt[3][8] = {};
        for (size_t q = q0; q < q0 + 8; ++q) {
            const CherryLane& L = S.lane[q];
            if (L.c < 0) continue;
            cnt[0][L.c & 7]++;
            for (int k = 0; k < 2; ++k)
                if (L.e[k] >= 0) cnt[1 + k][L.e[k] & 7]++;
        }
        for (size_t q = q0; q < q0 + 8; ++q) {
            const CherryLane& L = S.lane[q];
            uint32_t xr[3], gr[3];
            unsigned taken = 0;  // bank groups of this lane's dummy rows (distinct positions)
            auto dummy = [&](int acc) {
                int r = -1;
                for (int x = 0; x < 8; ++x)
                    if (!(taken >> x & 1u) && (r < 0 || cnt[acc][x] < cnt[acc][r])) r = x;
                taken |= 1u << r;
                cnt[acc][r]++;
                xr[acc] = (uint32_t)(npad + r);
                int row = r;
                if (distinct) {
                    while (step_used[row >> 6] >> (row & 63) & 1u) row += 8;  // (< 256: at most 96 per step)
                    step_used[row >> 6] |= 1ull << (row & 63);
                    R.n_spare = std::max(R.n_spare, (row + 8) & ~7);
                }
                gr[acc] = (uint32_t)(K * npad + row);
            };
            if (L.c >= 0) {
                xr[0] = (uint32_t)L.c;
                gr[0] = (uint32_t)(L.kc * npad + L.c);
            } else {
                dummy(0);
            }
            float cA[2], cB[2], cC[2], r0[2], dsv[2];
            bool hbk[2] = {false, false};
            for (int k = 0; k < 2; ++k) {
                if (L.c >= 0 && L.e[k] >= 0) {
                    xr[1 + k] = (uint32_t)L.e[k];
                    gr[1 + k] = (uint32_t)(L.ke[k] * npad + L.e[k]);
                    const float4 t = tp[ptp[L.p[k]]];  // (cA, cB, r0, n)
                    const bool hb = t.w > 8.f;        // 12-10 pair: its s^-10 coefficient goes to cC
                    cA[k] = t.x;
                    cB[k] = hb ? 0.f : -t.y;  // negated: pair_term2 takes -cB, -cC (no negations in the loop)
                    cC[k] = hb ? -t.y : 0.f;
                    hbk[k] = hb;
                    r0[k] = t.z;
                    dsv[k] = pdsv[L.p[k]];
                } else {
                    dummy(1 + k);
                    cA[k] = cB[k] = cC[k] = 0.f;
                    r0[k] = 1.f;
                    dsv[k] = 0.f;
                }
            }
            uint32_t d0, d1;
            memcpy(&d0, &dsv[0], 4);
            memcpy(&d1, &dsv[1], 4);
            // a.y bits 24-26: the centre / end 0 / end 1 is empty (PK_PRED: the kernel skips its store)
            const uint32_t fl = (L.c < 0 ? 1u : 0u) | (L.c < 0 || L.e[0] < 0 ? 2u : 0u) | (L.c < 0 || L.e[1] < 0 ? 4u : 0u);
            if (compact) {
                // a.x bits 24-25: pair k is a 12-10 (H-bond) pair, whose one nonzero dispersion
                // coefficient (-cC) then rides in b where a 12-6 pair's -cB goes (the kernel
                // rebuilds the (-cB, -cC) operands with selects: the same values, 8 B less)
                const uint32_t hbf = (hbk[0] ? 1u : 0u) | (hbk[1] ? 2u : 0u);
                R.a[q] = make_uint4(xr[0] | (xr[1] << 8) | (xr[2] << 16) | (hbf << 24),
                                    gr[0] | (gr[1] << 8) | (gr[2] << 16) | (fl << 24), d0, d1);
                R.b[q] = make_float4(cA[0], cA[1], hbk[0] ? cC[0] : cB[0], hbk[1] ? cC[1] : cB[1]);
                R.c2[q] = make_float2(r0[0], r0[1]);
            } else {
                R.a[q] = make_uint4(xr[0] | (xr[1] << 8) | (xr[2] << 16),
                                    gr[0] | (gr[1] << 8) | (gr[2] << 16) | (fl << 24), d0, d1);
                R.b[q] = make_float4(cA[0], cA[1], cB[0], cB[1]);
                R.c[q] = make_float4(r0[0], r0[1], cC[0], cC[1]);
            }
        }
    }
    return R;
}

// Owner-computes list: every contributor pair (i, j) becomes two directed
// entries (i <- j, primary) and (j <- i); entries are grouped by owner atom and
// the concatenated list is cut into 32 equal slices (lane l takes entries
// [l E, (l+1) E)), so every lane evaluates the same number of terms.  A lane
// flushes its register accumulator whenever its owner atom changes: the k-th
// flush of lane l goes to partial slot k*32 + l; comb/combidx list the slots of
// every atom for the final per-atom sum.
struct OwnerList {
    int E = 0, C = 0;
    std::vector<uint32_t> rec;  // [E][32]
    std::vector<float> dsv;     // [E][32]
    std::vector<int2> comb;     // [N]
    std::vector<uint16_t> combidx;
};

OwnerList build_owner(int n_atoms, const std::vector<int>& pi, const std::vector<int>& pj,
                      const std::vector<int>& ptp, const std::vector<float>& pdsv) {
    struct Ent { int a, b, tp; float dsv; int primary; };
    std::vector<std::vector<Ent>> lists(n_atoms);
    for (size_t q = 0; q < pi.size(); ++q) {
        lists[pi[q]].push_back({pi[q], pj[q], ptp[q], pdsv[q], 1});
        lists[pj[q]].push_back({pj[q], pi[q], ptp[q], pdsv[q], 0});
    }
    std::vector<Ent> flat;
    for (auto& l : lists) {
        std::sort(l.begin(), l.end(), [](const Ent& x, const Ent& y) { return x.b < y.b; });
        flat.insert(flat.end(), l.begin(), l.end());
    }
    OwnerList o;
    const int total = (int)flat.size();
    o.E = (total + 31) / 32;
    o.rec.assign((size_t)o.E * 32, 0u);
    o.dsv.assign((size_t)o.E * 32, 0.f);
    std::vector<std::vector<uint16_t>> slots(n_atoms);
    for (int l = 0; l < 32; ++l) {
        int k = 0;
        for (int t = 0; t < o.E; ++t) {
            const int idx = l * o.E + t;
            uint32_t fl;
            int a = 0, b = 0, tp = 0;
            float dv = 0.f;
            if (idx < total) {
                const Ent& e = flat[idx];
                a = e.a; b = e.b; tp = e.tp; dv = e.dsv;
                fl = e.primary ? OF_PRIMARY : 0;
                if (t == 0 || flat[idx - 1].a != a) fl |= OF_FIRST;
                if (t == o.E - 1 || idx == total - 1 || flat[idx + 1].a != a) {
                    fl |= OF_LAST;
                    slots[a].push_back((uint16_t)(k * 32 + l));
                    ++k;
                }
            } else {
                fl = OF_DUMMY | (t == 0 ? OF_FIRST : 0);
            }
            o.rec[(size_t)t * 32 + l] = (uint32_t)a | ((uint32_t)b << 8) | ((uint32_t)tp << 16) | (fl << 24);
            o.dsv[(size_t)t * 32 + l] = dv;
        }
        o.C = std::max(o.C, k);
    }
    o.comb.resize(n_atoms);
    for (int a = 0; a < n_atoms; ++a) {
        o.comb[a] = make_int2((int)o.combidx.size(), (int)slots[a].size());
        o.combidx.insert(o.combidx.end(), slots[a].begin(), slots[a].end());
    }
    return o;
}

// Hybrid list: every pair once, oriented owner i = min(i, j).  The owner-sorted
// list is cut into 32 equal slices (one per lane); a lane walks its slice run by
// run (a run = consecutive pairs with the same owner), keeps the owner's force in
// registers and stores one partial per run (slot k*32 + lane, like the owner list).
// The partner side is a read-modify-write of gradient slot s of atom j, with the
// (slot, j) targets of the 64 pairs of a step distinct (no atomics, one
// __syncwarp per step).  Steps are packed greedily per lane from its current run
// (pairs of a run can be taken in any order); a lane with no fitting pair gets an
// empty place (i == j == d, slot K = the spare row, flag OF_DUMMY).
// Record: i | j<<8 | tp<<16 | slot<<24 (4 bits) | flags<<28 (OF_FIRST, OF_LAST, OF_DUMMY).
struct HybridList {
    int S = 0, K = 1, C = 0;
    std::vector<uint32_t> rec;  // [S][2][32]
    std::vector<float> dsv;
    std::vector<int2> comb;
    std::vector<uint16_t> combidx;
};

HybridList build_hybrid_k(int n_atoms, const std::vector<int>& pi, const std::vector<int>& pj,
                          const std::vector<int>& ptp, const std::vector<float>& pdsv, int K) {
    struct Pr { int i, j, tp; float dsv; };
    std::vector<Pr> L;
    for (size_t q = 0; q < pi.size(); ++q)
        L.push_back({std::min(pi[q], pj[q]), std::max(pi[q], pj[q]), ptp[q], pdsv[q]});
    std::sort(L.begin(), L.end(), [](const Pr& a, const Pr& b) { return a.i != b.i ? a.i < b.i : a.j < b.j; });
    const int P = (int)L.size();
    const int per = (P + 31) / 32;
    // per lane: list of runs, each a vector of pairs
    std::vector<std::vector<std::vector<Pr>>> runs(32);
    for (int l = 0; l < 32; ++l)
        for (int t = l * per; t < std::min(P, (l + 1) * per); ++t) {
            if (runs[l].empty() || runs[l].back().front().i != L[t].i) runs[l].push_back({});
            runs[l].back().push_back(L[t]);
        }
    struct LaneState { size_t run = 0; bool started = false; int flushes = 0; };
    std::vector<LaneState> st(32);
    HybridList h;
    h.K = K;
    std::vector<std::vector<uint16_t>> slots(n_atoms);
    auto busy = [&](int l) { return st[l].run < runs[l].size(); };
    std::vector<int> cnt(n_atoms);
    while (true) {
        bool any = false;
        for (int l = 0; l < 32; ++l) any |= busy(l);
        if (!any) break;
        std::fill(cnt.begin(), cnt.end(), 0);
        const size_t base = h.rec.size();
        h.rec.resize(base + 64, 0u);
        h.dsv.resize(base + 64, 0.f);
        for (int u = 0; u < 2; ++u) {
            unsigned used[4] = {0, 0, 0, 0};  // j residues per quarter-warp
            for (int l = 0; l < 32; ++l) {
                uint32_t rec = 0;
                float dv = 0.f;
                int pick = -1;
                if (busy(l)) {
                    std::vector<Pr>& run = runs[l][st[l].run];
                    int fallback = -1;
                    for (size_t c = 0; c < run.size(); ++c) {
                        if (cnt[run[c].j] >= K) continue;
                        if (!(used[l / 8] >> (run[c].j & 7) & 1u)) { pick = (int)c; break; }
                        if (fallback < 0) fallback = (int)c;
                    }
                    if (pick < 0) pick = fallback;
                    if (pick >= 0) {
                        const Pr pr = run[pick];
                        run.erase(run.begin() + pick);
                        uint32_t fl = 0;
                        if (!st[l].started) { fl |= OF_FIRST; st[l].started = true; }
                        if (run.empty()) {
                            fl |= OF_LAST;
                            slots[pr.i].push_back((uint16_t)(st[l].flushes * 32 + l));
                            st[l].flushes++;
                            st[l].run++;
                            st[l].started = false;
                        }
                        rec = (uint32_t)pr.i | ((uint32_t)pr.j << 8) | ((uint32_t)pr.tp << 16) |
                              ((uint32_t)cnt[pr.j] << 24) | (fl << 28);
                        cnt[pr.j]++;
                        used[l / 8] |= 1u << (pr.j & 7);
                        dv = pr.dsv;
                    }
                }
                if (pick < 0) {  // empty place: spare row, a residue unused in the quarter if possible
                    unsigned d = 0;
                    while (d < 8 && d < (unsigned)n_atoms && (used[l / 8] >> d & 1u)) ++d;
                    if (d >= 8 || d >= (unsigned)n_atoms) d = 0;
                    used[l / 8] |= 1u << d;
                    rec = d | (d << 8) | ((uint32_t)K << 24) | ((uint32_t)OF_DUMMY << 28);
                }
                h.rec[base + (size_t)u * 32 + l] = rec;
                h.dsv[base + (size_t)u * 32 + l] = dv;
            }
        }
        h.S++;
    }
    for (int l = 0; l < 32; ++l) h.C = std::max(h.C, st[l].flushes);
    h.comb.resize(n_atoms);
    for (int a = 0; a < n_atoms; ++a) {
        h.comb[a] = make_int2((int)h.combidx.size(), (int)slots[a].size());
        h.combidx.insert(h.combidx.end(), slots[a].begin(), slots[a].end());
    }
    return h;
}

HybridList build_hybrid(int n_atoms, const std::vector<int>& pi, const std::vector<int>& pj,
                        const std::vector<int>& ptp, const std::vector<float>& pdsv) {
    HybridList best;
    for (int K = 1; K <= 4; ++K) {
        HybridList h = build_hybrid_k(n_atoms, pi, pj, ptp, pdsv, K);
        if (K == 1 || h.S < best.S) best = std::move(h);
    }
    return best;
}

}  // namespace

// =========================================================================== ABI
extern "C" {

const char* ad_last_error(void) { return g_err.c_str(); }

int32_t ad_version(void) { return 1; }

int32_t ad_context_create(int32_t cuda_device, ad_context** out) {
    if (!out) return fail(AD_ERR_INVALID_ARG, "out is NULL");
    *out = nullptr;
    int n = 0;
    CUDA_TRY(cudaGetDeviceCount(&n));
    if (cuda_device < 0 || cuda_device >= n) return fail(AD_ERR_INVALID_ARG, "device %d not in [0,%d)", cuda_device, n);
    ad_context* ctx = new (std::nothrow) ad_context();
    if (!ctx) return fail(AD_ERR_OOM, "host allocation failed");
    ctx->device = cuda_device;
    if (const char* m = getenv("AD_PAIRS_SMEM_MAX")) ctx->pairs_smem_max = atoi(m);
    if (const char* m = getenv("AD_PK_SMEM_MAX")) ctx->pk_smem_max = atoi(m);  // 0: no cherry schedules (A/B)
    if (const char* m = getenv("AD_INTRA_MODE"))
        ctx->intra_mode = strcmp(m, "owner") == 0 ? INTRA_OWNER : strcmp(m, "hybrid") == 0 ? INTRA_HYBRID : INTRA_SCATTER;
    cudaError_t e = cudaSetDevice(cuda_device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&ctx->n_sms, cudaDevAttrMultiProcessorCount, cuda_device);
    if (e == cudaSuccess)
        e = cudaDeviceGetAttribute(&ctx->max_smem_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, cuda_device);
    if (e == cudaSuccess)
        e = cudaDeviceGetAttribute(&ctx->smem_per_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, cuda_device);
    if (e == cudaSuccess) e = cudaMalloc(&ctx->d_err, sizeof(int32_t));
    if (e == cudaSuccess) e = cudaMemset(ctx->d_err, 0, sizeof(int32_t));
    if (e == cudaSuccess) e = cudaHostAlloc(reinterpret_cast<void**>(&ctx->h_err), sizeof(int32_t), cudaHostAllocMapped);
    if (e == cudaSuccess) *ctx->h_err = 0;
    if (e == cudaSuccess) e = cudaHostGetDevicePointer(reinterpret_cast<void**>(&ctx->d_err_seen), ctx->h_err, 0);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&ctx->err_ev, cudaEventDisableTiming);
    if (e != cudaSuccess) {
        delete ctx;
        return fail(AD_ERR_CUDA, "context init: %s", cudaGetErrorString(e));
    }
    *out = ctx;
    return AD_OK;
}

int32_t ad_context_destroy(ad_context* ctx) {
    if (!ctx) return AD_OK;
    cudaSetDevice(ctx->device);
    cudaDeviceSynchronize();
    for (auto& l : ctx->ligs) {
        if (l.d_base && l.d_base != l.d_blob) cudaFree(l.d_base);
        if (l.d_blob) cudaFree(l.d_blob);
    }
    if (ctx->d_tmap) cudaFree(ctx->d_tmap);
    if (ctx->d_ed) cudaFree(ctx->d_ed);
    if (ctx->d_ligtab) cudaFree(ctx->d_ligtab);
    if (ctx->d_err) cudaFree(ctx->d_err);
    if (ctx->h_err) cudaFreeHost(ctx->h_err);
    if (ctx->err_ev) cudaEventDestroy(ctx->err_ev);
    delete ctx;
    return AD_OK;
}

int32_t ad_upload_grids(ad_context* ctx, const ad_grid_desc* d, const float* maps, int32_t maps_on_device,
                        void* stream) {
    NvtxRange nvtx_range("ad_upload_grids");
    if (!ctx || !d || !maps) return fail(AD_ERR_INVALID_ARG, "null argument");
    if (d->nx < 2 || d->ny < 2 || d->nz < 2) return fail(AD_ERR_INVALID_ARG, "grid needs >= 2 points per axis");
    if (d->n_maps < 3 || d->n_maps > AD_MAX_MAPS) return fail(AD_ERR_LIMIT, "n_maps %d not in [3,%d]", d->n_maps, AD_MAX_MAPS);
    if (!(d->spacing > 0.f) || !std::isfinite(d->spacing)) return fail(AD_ERR_INVALID_ARG, "spacing must be > 0");
    const size_t plane = (size_t)d->nx * d->ny, vol = plane * d->nz;
    if (vol > (size_t)1 << 31) return fail(AD_ERR_LIMIT, "grid too large");
    if (int32_t rc = set_device(ctx)) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    std::vector<float> h(vol * d->n_maps);
    if (maps_on_device) {
        CUDA_TRY(cudaMemcpyAsync(h.data(), maps, sizeof(float) * h.size(), cudaMemcpyDeviceToHost, st));
        CUDA_TRY(cudaStreamSynchronize(st));
    } else {
        memcpy(h.data(), maps, sizeof(float) * h.size());
    }
    const int nt = d->n_maps - 2;
    const float* E = h.data() + (size_t)nt * vol;
    const float* D = h.data() + (size_t)(nt + 1) * vol;
    // Cell records (3 x 256-bit loads per atom, 8x the map bytes) up to 1 GiB of records,
    // else x-pair records (8 loads per atom, 2x bytes).  The poses of a search stay in the
    // pocket, so the cells they touch are a small part of the grid and L2-resident even
    // when the whole record set is not: config 3 (96^3, 8 type maps: 283 MB of cell
    // records) runs 104.7 (x-pair) -> 98.6 ms per LS launch with cells (its LS kernel is
    // L1-bound, and a cell gather is 3 wide loads instead of 8)
    const size_t cell_bytes = vol * ((size_t)nt * 32 + 64);
    int layout = cell_bytes <= ((size_t)1 << 30) ? 1 : 0;
    if (const char* e = getenv("AD_GRID_LAYOUT")) layout = strcmp(e, "cell") == 0 ? 1 : strcmp(e, "xpair") == 0 ? 0 : layout;
    if (ctx->d_tmap) { cudaFree(ctx->d_tmap); ctx->d_tmap = nullptr; }
    if (ctx->d_ed) { cudaFree(ctx->d_ed); ctx->d_ed = nullptr; }
    ctx->has_grid = false;
    GridDev& g = ctx->grid;
    g = GridDev{};
    if (layout == 1) {
        auto at = [&](const float* m, int x, int y, int z) {
            x = std::min(x, d->nx - 1); y = std::min(y, d->ny - 1); z = std::min(z, d->nz - 1);
            return m[((size_t)z * d->ny + y) * d->nx + x];
        };
        std::vector<float> tc((size_t)nt * vol * 8), edc(vol * 16);
        for (int z = 0; z < d->nz; ++z)
            for (int y = 0; y < d->ny; ++y)
                for (int x = 0; x < d->nx; ++x) {
                    const size_t cell = ((size_t)z * d->ny + y) * d->nx + x;
                    for (int c = 0; c < 8; ++c) {
                        const int dx = c & 1, dy = (c >> 1) & 1, dz = c >> 2;
                        for (int m = 0; m < nt; ++m)
                            tc[((size_t)m * vol + cell) * 8 + c] = at(h.data() + (size_t)m * vol, x + dx, y + dy, z + dz);
                        edc[cell * 16 + c] = at(E, x + dx, y + dy, z + dz);
                        edc[cell * 16 + 8 + c] = at(D, x + dx, y + dy, z + dz);
                    }
                }
        CUDA_TRY(cudaMalloc(&ctx->d_tmap, sizeof(float) * tc.size()));
        CUDA_TRY(cudaMalloc(&ctx->d_ed, sizeof(float) * edc.size()));
        CUDA_TRY(cudaMemcpy(ctx->d_tmap, tc.data(), sizeof(float) * tc.size(), cudaMemcpyHostToDevice));
        CUDA_TRY(cudaMemcpy(ctx->d_ed, edc.data(), sizeof(float) * edc.size(), cudaMemcpyHostToDevice));
        g.tc8 = (const float*)ctx->d_tmap;
        g.ed8 = (const float*)ctx->d_ed;
    } else {
        std::vector<float2> tm(vol * nt);
        std::vector<float4> ed(vol);
        for (int m = 0; m < nt; ++m)
            for (size_t zy = 0; zy < plane / d->nx * d->nz; ++zy)
                for (int x = 0; x < d->nx; ++x) {
                    const size_t i = zy * d->nx + x, i1 = zy * d->nx + std::min(x + 1, d->nx - 1);
                    tm[m * vol + i] = make_float2(h[m * vol + i], h[m * vol + i1]);
                }
        for (size_t zy = 0; zy < plane / d->nx * d->nz; ++zy)
            for (int x = 0; x < d->nx; ++x) {
                const size_t i = zy * d->nx + x, i1 = zy * d->nx + std::min(x + 1, d->nx - 1);
                ed[i] = make_float4(E[i], E[i1], D[i], D[i1]);
            }
        CUDA_TRY(cudaMalloc(&ctx->d_tmap, sizeof(float2) * tm.size()));
        CUDA_TRY(cudaMalloc(&ctx->d_ed, sizeof(float4) * ed.size()));
        CUDA_TRY(cudaMemcpy(ctx->d_tmap, tm.data(), sizeof(float2) * tm.size(), cudaMemcpyHostToDevice));
        CUDA_TRY(cudaMemcpy(ctx->d_ed, ed.data(), sizeof(float4) * ed.size(), cudaMemcpyHostToDevice));
        g.tmap = (const float2*)ctx->d_tmap;
        g.ed = (const float4*)ctx->d_ed;
    }
    g.layout = layout;
    g.nx = d->nx; g.ny = d->ny; g.nz = d->nz; g.n_type = nt;
    g.ox = d->origin[0]; g.oy = d->origin[1]; g.oz = d->origin[2];
    g.h = d->spacing;
    g.inv_h = 1.0f / d->spacing;
    ctx->grid_n_type = nt;
    ctx->has_grid = true;
    return AD_OK;
}

int32_t ad_upload_ligand(ad_context* ctx, const ad_ligand_desc* d, ad_ligand_id* out) {
    NvtxRange nvtx_range("ad_upload_ligand");
    if (!ctx || !d || !out) return fail(AD_ERR_INVALID_ARG, "null argument");
    *out = -1;
    if (!ctx->has_grid) return fail(AD_ERR_STATE, "upload grids before ligands");
    const int N = d->n_atoms, T = d->n_tors, P = d->n_pairs, nt = d->n_types;
    if (N < 1 || N > AD_MAX_ATOMS) return fail(AD_ERR_LIMIT, "n_atoms %d not in [1,%d]", N, AD_MAX_ATOMS);
    if (T < 0 || T > AD_MAX_TORS) return fail(AD_ERR_LIMIT, "n_tors %d not in [0,%d]", T, AD_MAX_TORS);
    if (nt < 1 || nt > AD_MAX_TYPES) return fail(AD_ERR_LIMIT, "n_types %d not in [1,%d]", nt, AD_MAX_TYPES);
    if (P < 0) return fail(AD_ERR_INVALID_ARG, "n_pairs < 0");
    if (!d->ref_xyz || !d->atom_map || !d->atom_type || !d->charge || !d->tp_coef || !d->type_S || !d->type_V ||
        !d->ff || (T && (!d->tors_axis || !d->tors_moving)) || (P && !d->pairs))
        return fail(AD_ERR_INVALID_ARG, "null array in ligand descriptor");
    for (int a = 0; a < N; ++a) {
        if (d->atom_map[a] < 0 || d->atom_map[a] >= ctx->grid_n_type)
            return fail(AD_ERR_INVALID_ARG, "atom_map[%d]=%d not a type map", a, d->atom_map[a]);
        if (d->atom_type[a] < 0 || d->atom_type[a] >= nt)
            return fail(AD_ERR_INVALID_ARG, "atom_type[%d]=%d out of range", a, d->atom_type[a]);
    }
    // --- torsion tree from the moving sets (must be laminar, listed root -> leaf)
    std::vector<std::vector<uint8_t>> M(T, std::vector<uint8_t>(N));
    std::vector<int> msize(T, 0);
    for (int b = 0; b < T; ++b) {
        for (int a = 0; a < N; ++a) {
            M[b][a] = d->tors_moving[(size_t)b * N + a] ? 1 : 0;
            msize[b] += M[b][a];
        }
        const int a0 = d->tors_axis[2 * b], c0 = d->tors_axis[2 * b + 1];
        if (a0 < 0 || a0 >= N || c0 < 0 || c0 >= N || a0 == c0)
            return fail(AD_ERR_INVALID_ARG, "torsion %d axis atoms out of range", b);
        if (M[b][a0] || !M[b][c0])
            return fail(AD_ERR_INVALID_ARG, "torsion %d: need a not moving and c moving", b);
    }
    std::vector<int> parent(T, -1);
    for (int b = 0; b < T; ++b) {
        for (int b2 = 0; b2 < T; ++b2) {
            if (b2 == b) continue;
            int inter = 0;
            for (int a = 0; a < N; ++a) inter += M[b][a] & M[b2][a];
            const bool sub = inter == msize[b], sup = inter == msize[b2], dis = inter == 0;
            if (!sub && !sup && !dis) return fail(AD_ERR_INVALID_ARG, "moving sets of torsions %d and %d overlap", b, b2);
            if (sub && msize[b] == msize[b2]) return fail(AD_ERR_INVALID_ARG, "torsions %d and %d move the same atoms", b, b2);
            if (sub && b2 > b) return fail(AD_ERR_INVALID_ARG, "torsion %d listed before its parent %d (need root->leaf)", b, b2);
            // every other torsion moves both axis atoms of b or neither
            const int a0 = d->tors_axis[2 * b], c0 = d->tors_axis[2 * b + 1];
            if (M[b2][a0] != M[b2][c0])
                return fail(AD_ERR_INVALID_ARG, "torsion %d moves only one axis atom of torsion %d", b2, b);
            if (sub && (parent[b] < 0 || msize[b2] < msize[parent[b]])) parent[b] = b2;
        }
    }
    // --- DFS order: root atoms, then each torsion subtree (children in index order)
    std::vector<int> order;
    order.reserve(N);
    std::vector<int> lo(T), hi(T);
    std::vector<std::vector<int>> kids(T + 1);  // kids[T] = top level
    for (int b = 0; b < T; ++b) kids[parent[b] < 0 ? T : parent[b]].push_back(b);
    std::vector<int> owner(N, -1);  // deepest torsion moving the atom
    for (int a = 0; a < N; ++a) {
        int best = -1;
        for (int b = 0; b < T; ++b)
            if (M[b][a] && (best < 0 || msize[b] < msize[best])) best = b;
        owner[a] = best;
    }
    struct Frame { int node; size_t next; };
    std::vector<Frame> stack;
    for (int a = 0; a < N; ++a)
        if (owner[a] < 0) order.push_back(a);
    for (int top : kids[T]) {
        stack.push_back({top, 0});
        lo[top] = (int)order.size();
        for (int a = 0; a < N; ++a)
            if (owner[a] == top) order.push_back(a);
        while (!stack.empty()) {
            Frame& f = stack.back();
            if (f.next < kids[f.node].size()) {
                const int c = kids[f.node][f.next++];
                lo[c] = (int)order.size();
                for (int a = 0; a < N; ++a)
                    if (owner[a] == c) order.push_back(a);
                stack.push_back({c, 0});
            } else {
                hi[f.node] = (int)order.size();
                stack.pop_back();
            }
        }
    }
    if ((int)order.size() != N) return fail(AD_ERR_INVALID_ARG, "internal: DFS order incomplete");
    std::vector<int> newi(N);
    for (int k = 0; k < N; ++k) newi[order[k]] = k;
    for (int b = 0; b < T; ++b)
        if (hi[b] - lo[b] != msize[b]) return fail(AD_ERR_INVALID_ARG, "internal: moving set %d not contiguous", b);

    // --- per-type-pair table
    std::vector<float4> tp((size_t)nt * nt);
    for (int t = 0; t < nt * nt; ++t) {
        const float* c = d->tp_coef + 5 * t;
        if (c[3] != 12.f || (c[4] != 6.f && c[4] != 10.f))
            return fail(AD_ERR_INVALID_ARG, "tp_coef entry %d: exponents (%g,%g) unsupported (need 12-6 or 12-10)", t,
                        c[3], c[4]);
        tp[t] = make_float4(c[0], c[1], c[2], c[4]);
    }
    const ad_ff_params& F = *d->ff;
    // --- pairs (new numbering) with desolvation prefactors
    std::vector<int> pi(P), pj(P), ptp(P);
    std::vector<float> pd(P), pcq(P);
    for (int q = 0; q < P; ++q) {
        const int i = d->pairs[2 * q], j = d->pairs[2 * q + 1];
        if (i < 0 || i >= N || j < 0 || j >= N || i == j) return fail(AD_ERR_INVALID_ARG, "pair %d = (%d,%d) invalid", q, i, j);
        pi[q] = newi[i];
        pj[q] = newi[j];
        const int ti = d->atom_type[i], tj = d->atom_type[j];
        ptp[q] = ti * nt + tj;
        const double qi = std::fabs((double)d->charge[i]), qj = std::fabs((double)d->charge[j]);
        pd[q] = (float)((double)F.coeff_ds * (((double)d->type_S[ti] + (double)F.qasp * qi) * (double)d->type_V[tj] +
                                              ((double)d->type_S[tj] + (double)F.qasp * qj) * (double)d->type_V[ti]));
        pcq[q] = (float)((double)F.coeff_el * (double)d->charge[i] * (double)d->charge[j]);
    }
    if (nt * nt > 256) return fail(AD_ERR_LIMIT, "n_types^2 > 256");
    const int mode = ctx->intra_mode;
    std::vector<int> slot(N);  // storage slot (X / gradient row) of every atom; identity unless balanced
    for (int k = 0; k < N; ++k) slot[k] = k;
    Schedule sch;
    OwnerList own;
    CherrySchedule cs;
    bool cherry = false, cherry_gm = false;
    if (mode == INTRA_OWNER) {
        own = build_owner(N, pi, pj, ptp, pd);
        if (own.C * 32 > 65535) return fail(AD_ERR_LIMIT, "too many owner chunks");
        sch.rounds = 0;
        sch.slots = 1;
        sch.rec = own.rec;
        sch.dsv = own.dsv;
    } else if (mode == INTRA_HYBRID) {
        HybridList hy = build_hybrid(N, pi, pj, ptp, pd);
        if (hy.C * 32 > 65535) return fail(AD_ERR_LIMIT, "too many hybrid runs");
        sch.rounds = hy.S;
        sch.slots = hy.K;
        sch.rec = std::move(hy.rec);
        sch.dsv = std::move(hy.dsv);
        own.C = hy.C;
        own.comb = std::move(hy.comb);
        own.combidx = std::move(hy.combidx);
    } else {
        slot = balance_slots(N, pi, pj);
        std::vector<int> si(P), sj(P);
        for (int q = 0; q < P; ++q) {
            si[q] = slot[pi[q]];
            sj[q] = slot[pj[q]];
        }
        // the cherry schedule when it fits shared memory (its records and the prec
        // list) and its row offsets fit 16 bits; else the pair-step schedule
        // A cherry schedule too long for shared memory streams its records from global
        // memory instead (cherry_gm: intra_cherry_gm, 128-register kernels); the 8-bit
        // row indices cap the gradient slots (cherry_max_slots).  AD_PK_SMEM_MAX=0 turns
        // cherries off altogether, AD_CHERRY_GM=0 the global-memory variant (A/B knobs).
        static const bool gm_on = !getenv("AD_CHERRY_GM") || atoi(getenv("AD_CHERRY_GM")) != 0;
        const int max_K = cherry_max_slots(npad_of(N));
        if (ctx->pk_smem_max > 0 && P > 0 && max_K > 0) {
            const int max_steps = std::min(ctx->pairs_smem_max / (kPairsPerStep * 12), ctx->pk_smem_max / (kLanes * 48));
            cs = schedule_cherries(npad_of(N), si, sj, ctx->sched_effort, gm_on ? (1 << 30) : max_steps, max_K);
            const bool fit = cherry_rows_fit(npad_of(N), cs.slots);
            cherry = cs.steps <= max_steps && fit;
            cherry_gm = !cherry && fit && gm_on;
        }
        // the prec list (the paper-style baseline's pairs; the warp engine's schedule
        // when it runs no cherries) is the pair-step schedule either way, so the
        // baseline is the same program with or without cherries
        sch = schedule_pairs(N, si, sj, ptp, pd, pcq, ctx->sched_effort);
        if (cherry && (int64_t)(sch.rec.size() + sch.dsv.size()) * 4 > ctx->pairs_smem_max) {
            cherry = false;
            cherry_gm = gm_on;
        }
    }
    if (own.comb.empty()) own.comb.assign(N, make_int2(0, 0));

    // --- atoms, chains, masks (new numbering)
    std::vector<float4> atoms(N);
    std::vector<int2> info(N);
    std::vector<uint8_t> chain;
    std::vector<uint2> mask(N);
    for (int k = 0; k < N; ++k) {
        const int a = order[k];
        atoms[k] = make_float4(d->ref_xyz[3 * a], d->ref_xyz[3 * a + 1], d->ref_xyz[3 * a + 2], d->charge[a]);
        std::vector<int> ch;
        uint64_t m = 0;
        for (int b = 0; b < T; ++b)
            if (M[b][a]) { ch.push_back(b); m |= 1ull << b; }
        std::sort(ch.begin(), ch.end(), [&](int x, int y) { return msize[x] < msize[y]; });  // leaf -> root
        info[k] = make_int2(d->atom_map[a] | (d->atom_type[a] << 8) | ((int)ch.size() << 16) | (slot[k] << 24),
                            (int)chain.size());
        for (int b : ch) chain.push_back((uint8_t)b);
        mask[k] = make_uint2((uint32_t)m, (uint32_t)(m >> 32));
    }
    std::vector<float4> tors(2 * std::max(T, 1));
    std::vector<double> tors64(6 * std::max(T, 1));
    std::vector<int4> tinfo(std::max(T, 1));
    for (int b = 0; b < T; ++b) {
        const int a0 = d->tors_axis[2 * b], c0 = d->tors_axis[2 * b + 1];
        const double P0[3] = {d->ref_xyz[3 * a0], d->ref_xyz[3 * a0 + 1], d->ref_xyz[3 * a0 + 2]};
        double u[3] = {d->ref_xyz[3 * c0] - P0[0], d->ref_xyz[3 * c0 + 1] - P0[1], d->ref_xyz[3 * c0 + 2] - P0[2]};
        const double nu = std::sqrt(u[0] * u[0] + u[1] * u[1] + u[2] * u[2]);
        if (!(nu > 0)) return fail(AD_ERR_INVALID_ARG, "torsion %d has a zero-length axis", b);
        tors[2 * b] = make_float4((float)P0[0], (float)P0[1], (float)P0[2], 0.f);
        tors[2 * b + 1] = make_float4((float)(u[0] / nu), (float)(u[1] / nu), (float)(u[2] / nu), 0.f);
        for (int k = 0; k < 3; ++k) {
            tors64[6 * b + k] = P0[k];
            tors64[6 * b + 3 + k] = u[k] / nu;
        }
        tinfo[b] = make_int4(slot[newi[a0]], slot[newi[c0]], lo[b], hi[b]);
    }

    LigHeader H{};
    H.n_atoms = N; H.n_tors = T; H.n_pairs = P; H.n_types = nt;
    H.n_rounds = sch.rounds;  // per blob below
    H.n_slots = sch.slots;
    H.n_chain = (int)chain.size();
    H.n_pad = npad_of(N);  // gradient-slot row stride
    H.intra_mode = mode;
    H.n_entries = own.E;
    H.n_chunks = own.C;
    const double sig = F.sigma_ds;
    H.ff[FF_DELTA] = 0.5f * F.smooth;
    H.ff[FF_CUT_VDW] = F.cut_vdw;
    H.ff[FF_CUT_EL] = F.cut_el;
    H.ff[FF_EL_RMIN] = F.el_rmin;
    H.ff[FF_DIEL_A] = F.diel_A;
    H.ff[FF_DIEL_B] = F.diel_B;
    H.ff[FF_DIEL_K] = F.diel_k;
    H.ff[FF_DIEL_LB] = (float)((double)F.diel_lambda * (double)F.diel_B);
    H.ff[FF_COEFF_EL] = F.coeff_el;
    H.ff[FF_DS_EXP2] = (float)(-1.4426950408889634 / (2.0 * sig * sig));
    H.ff[FF_INV_S2] = (float)(1.0 / (sig * sig));
    H.ff[FF_W_OUT] = F.w_out;
    // Two blobs when the warp engine runs a cherry schedule: the warp engine's (tables +
    // cherry records; no pair-step list, no type-pair table) and the paper-style
    // baseline's (tables + type-pair table + the pair-step list), so neither stages
    // bytes it never reads.  Otherwise one blob serves both engines.
    if (const char* dump = getenv("AD_DUMP_SCHEDULE")) {  // debugging aid: raw schedule records
        if (FILE* f = fopen(dump, "ab")) {
            const int32_t hdr[4] = {N, sch.rounds, sch.slots, H.n_pad};
            fwrite(hdr, sizeof(hdr), 1, f);
            fwrite(sch.rec.data(), sizeof(uint32_t), sch.rec.size(), f);
            fclose(f);
        }
    }
    if (cherry && (int64_t)(sch.rec.size() + sch.dsv.size()) * 4 > ctx->pairs_smem_max)
        return fail(AD_ERR_STATE, "internal: cherry schedule with a global-memory prec list");
    struct Built {
        std::vector<unsigned char> buf;
        LigHeader h;
        WarpScratch ws;
    };
    auto build_blob = [&](bool warp_cherry) {
        Built o;
        LigHeader& h = o.h;
        h = H;
        h.n_rounds = warp_cherry ? cs.steps : sch.rounds;
        h.n_slots = warp_cherry ? cs.slots : sch.slots;
        h.base_rounds = sch.rounds;
        h.base_slots = sch.slots;
        BlobBuilder B;
        B.put(&h, sizeof(h));
        h.off_atoms = B.put(atoms.data(), sizeof(float4) * N);
        h.off_info = B.put(info.data(), sizeof(int2) * N);
        h.off_tors = B.put(tors.data(), sizeof(float4) * 2 * T);
        h.off_tors64 = B.put(tors64.data(), sizeof(double) * 6 * T);
        h.off_tinfo = B.put(tinfo.data(), sizeof(int4) * T);
        h.off_chain = B.put(chain.data(), chain.size());
        h.off_mask = B.put(mask.data(), sizeof(uint2) * N);
        h.off_comb = B.put(own.comb.data(), sizeof(int2) * own.comb.size());
        h.off_combidx = B.put(own.combidx.data(), sizeof(uint16_t) * own.combidx.size());
        o.ws = warp_scratch_layout(N, T, h.n_slots, own.C);
        if (warp_cherry) {
            // cherry records (ad_internal.h pka / pkb / pkc), staged with the tables (or,
            // cherry_gm, left in global memory).  Distinct dummy rows when they fit the
            // 8-bit row indices and at most 32 spare rows (512 B per warp), else shared
            // dummies with predicated stores (PK_PRED).
            CherryRecords cr = pack_cherries(cs, h.n_pad, ptp, tp, pd, true, cherry_gm);
            h.pk_flags = cherry_gm ? PK_GMEM : 0;
            // (global-memory cherries always take the predicated loop: measured faster than
            // distinct dummies on config 3, 114.1 vs 120.4 ms per LS launch)
            if (cherry_gm || cs.slots * h.n_pad + cr.n_spare > 256 || cr.n_spare > 32) {
                cr = pack_cherries(cs, h.n_pad, ptp, tp, pd, false, cherry_gm);
                h.pk_flags |= PK_PRED;
            }
            o.ws = warp_scratch_layout(N, T, h.n_slots, own.C, cr.n_spare);
            h.off_tp = h.off_prec = h.off_pdsv = h.off_pkg = 0;
            h.off_pk = B.put(cr.a.data(), sizeof(uint4) * cr.a.size());
            B.put(cr.b.data(), sizeof(float4) * cr.b.size());
            if (cherry_gm) B.put(cr.c2.data(), sizeof(float2) * cr.c2.size());
            else B.put(cr.c.data(), sizeof(float4) * cr.c.size());
            h.pairs_gmem = cherry_gm ? 1 : 0;  // (cherry_gm: records after the staged prefix)
            h.blob_bytes = (int32_t)B.buf.size();
            h.stage_bytes = cherry_gm ? h.off_pk : h.blob_bytes;
        } else {
            // 8 copies of every entry, copy c at index t*8 + c: lane l reads copy l % 8,
            // so the 8 lanes of a quarter-warp always hit 8 different bank groups.
            std::vector<float4> tp8(tp.size() * AD_TP_COPIES);
            for (size_t t = 0; t < tp.size(); ++t)
                for (int c = 0; c < AD_TP_COPIES; ++c) tp8[t * AD_TP_COPIES + c] = tp[t];
            h.off_tp = B.put(tp8.data(), sizeof(float4) * tp8.size());
            // the pair schedule goes last: large schedules stay in global memory (read
            // through L1, one copy per SM) instead of being staged into every CTA
            h.off_prec = B.put(sch.rec.data(), sizeof(uint32_t) * sch.rec.size());
            h.off_pdsv = B.put(sch.dsv.data(), sizeof(float) * sch.dsv.size());
            h.off_pk = 0;
            h.off_pkg = 0;
            h.pairs_gmem = (int32_t)B.buf.size() - h.off_prec > ctx->pairs_smem_max ? 1 : 0;
            static const bool pkg_on = !getenv("AD_PKG") || atoi(getenv("AD_PKG")) != 0;  // A/B knob
            if (h.pairs_gmem && pkg_on && h.intra_mode == INTRA_SCATTER &&
                o.ws.g + 16 * (h.n_pad * (h.n_slots + 1)) <= 0xffff) {
                // pre-decoded places for the global-memory pair loop (intra_packed_gm),
                // after the prec list (never staged; the baseline keeps reading prec)
                const int n_places = (int)sch.rec.size();
                const uint32_t npad = (uint32_t)h.n_pad;
                std::vector<uint4> pka(n_places);
                std::vector<float2> pkb(n_places);
                for (int q = 0; q < n_places; ++q) {
                    const uint32_t rec = sch.rec[q];
                    const uint32_t i = rec & 0xffu, j = (rec >> 8) & 0xffu, si = (rec >> 16) & 0xfu, sj = (rec >> 20) & 0xfu;
                    const uint32_t gi = (uint32_t)o.ws.g + 16u * (si * npad + i);
                    const uint32_t gj = (uint32_t)o.ws.g + 16u * (sj * npad + j);
                    if ((int)si == sch.slots) {  // empty place: zero-charge rows, zero coefficients, spare row
                        // bit 15 of the i offset marks the empty place (X offsets < 2^13)
                        pka[q] = make_uint4((16u * npad) | 0x8000u | ((16u * (npad + 1)) << 16), gi | (gj << 16), 0u, 0u);
                        pkb[q] = make_float2(0.f, 1.f);
                        continue;
                    }
                    const float4 c = tp[rec >> 24];
                    uint32_t ud, ua;
                    memcpy(&ud, &sch.dsv[2 * q], 4);
                    memcpy(&ua, &c.x, 4);
                    pka[q] = make_uint4((16u * i) | ((16u * j) << 16), gi | (gj << 16), ud, ua);
                    pkb[q] = make_float2(c.y, c.w > 8.f ? -c.z : c.z);  // sign bit = 12-10 (H-bond) pair
                }
                h.off_pkg = B.put(pka.data(), sizeof(uint4) * pka.size());
                B.put(pkb.data(), sizeof(float2) * pkb.size());
            }
            h.blob_bytes = (int32_t)B.buf.size();
            h.stage_bytes = h.pairs_gmem ? h.off_prec : h.blob_bytes;
        }
        h.scratch_bytes = o.ws.bytes;
        h.ws_g = o.ws.g; h.ws_w = o.ws.w; h.ws_d = o.ws.d; h.ws_trig = o.ws.trig; h.ws_trig64 = o.ws.trig64;
        h.ws_tw = o.ws.tw; h.ws_genes = o.ws.genes; h.ws_part = o.ws.part;
        memcpy(B.buf.data(), &h, sizeof(h));
        o.buf = std::move(B.buf);
        return o;
    };
    const Built base = build_blob(false);
    Built warp;
    const bool two = cherry || cherry_gm;
    if (two) warp = build_blob(true);
    const Built& W = two ? warp : base;

    std::lock_guard<std::mutex> lock(ctx->mu);
    if (int32_t rc = set_device(ctx)) return rc;
    LigSlot s;
    s.blob_bytes = W.h.stage_bytes;     // shared-memory bytes staged per CTA (warp engine)
    s.base_bytes = base.h.stage_bytes;  // ... (paper-style baseline)
    s.scratch_bytes = W.ws.bytes;
    s.scratch_simt = W.ws.bytes_simt;
    s.block_scratch = block_scratch_layout(N, T, 0).bytes;
    s.n_atoms = N;
    s.n_tors = T;
    s.pkg = (W.h.off_pkg != 0 && 6 + T > 32) || (W.h.pk_flags & PK_GMEM);  // runs on the 128-register kernels
    s.smem_cherry = W.h.intra_mode == INTRA_SCATTER && W.h.off_pk != 0 && !(W.h.pk_flags & (PK_GMEM | PK_PRED));
    s.gm_cherry = W.h.intra_mode == INTRA_SCATTER && W.h.off_pk != 0 && (W.h.pk_flags & PK_GMEM);
    memcpy(s.ff, H.ff, sizeof(s.ff));
    CUDA_TRY(cudaMalloc(&s.d_blob, W.buf.size()));
    CUDA_TRY(cudaMemcpy(s.d_blob, W.buf.data(), W.buf.size(), cudaMemcpyHostToDevice));
    s.d_base = s.d_blob;
    if (two) {
        if (cudaMalloc(&s.d_base, base.buf.size()) != cudaSuccess) {
            cudaFree(s.d_blob);
            return fail(AD_ERR_OOM, "ligand blob allocation failed");
        }
        CUDA_TRY(cudaMemcpy(s.d_base, base.buf.data(), base.buf.size(), cudaMemcpyHostToDevice));
    }
    s.live = true;
    // the lowest free id (ids of freed ligands are reused), else a new one
    int id = 0;
    while (id < (int)ctx->ligs.size() && ctx->ligs[id].live) ++id;
    if (id >= AD_MAX_LIGANDS) {
        if (s.d_base != s.d_blob) cudaFree(s.d_base);
        cudaFree(s.d_blob);
        return fail(AD_ERR_LIMIT, "too many ligands");
    }
    if (id == (int)ctx->ligs.size()) ctx->ligs.push_back(s); else ctx->ligs[id] = s;
    if (int32_t rc = sync_ligtab(ctx, id)) return rc;
    *out = (ad_ligand_id)id;
    return AD_OK;
}

int32_t ad_free_ligand(ad_context* ctx, ad_ligand_id lig) {
    if (!ctx) return fail(AD_ERR_INVALID_ARG, "ctx is NULL");
    std::lock_guard<std::mutex> lock(ctx->mu);
    if (lig < 0 || lig >= (int)ctx->ligs.size() || !ctx->ligs[lig].live)
        return fail(AD_ERR_INVALID_ARG, "bad ligand id %d", lig);
    if (int32_t rc = set_device(ctx)) return rc;
    CUDA_TRY(cudaDeviceSynchronize());
    if (ctx->ligs[lig].d_base != ctx->ligs[lig].d_blob) cudaFree(ctx->ligs[lig].d_base);
    cudaFree(ctx->ligs[lig].d_blob);
    ctx->ligs[lig] = LigSlot{};
    return sync_ligtab(ctx, lig);
}

int32_t ad_set_launch_ligands(ad_context* ctx, const int32_t* ids, int32_t n) {
    if (!ctx) return fail(AD_ERR_INVALID_ARG, "ctx is NULL");
    if (n < 0 || (n > 0 && !ids)) return fail(AD_ERR_INVALID_ARG, "bad launch ligand list");
    std::lock_guard<std::mutex> lock(ctx->mu);
    for (int32_t k = 0; k < n; ++k)
        if (ids[k] < 0 || ids[k] >= (int)ctx->ligs.size() || !ctx->ligs[ids[k]].live)
            return fail(AD_ERR_INVALID_ARG, "launch ligand %d (entry %d) is not a live ligand", ids[k], k);
    ctx->launch_set.assign(ids, ids + n);
    return AD_OK;
}

int32_t ad_set_schedule_effort(ad_context* ctx, int32_t effort) {
    if (!ctx) return fail(AD_ERR_INVALID_ARG, "ctx is NULL");
    if (effort < 0 || effort > 2) return fail(AD_ERR_INVALID_ARG, "schedule effort %d not in 0..2", effort);
    std::lock_guard<std::mutex> lock(ctx->mu);
    ctx->sched_effort = effort;
    return AD_OK;
}

}  // extern "C"

// --------------------------------------------------------------- launches
namespace {

typedef void (*WarpKernelFn)(const KParams);
struct WarpKernel {
    WarpKernelFn lo, hi;  // register budgets AD_WARP_MAXNREG / AD_WARP_MAXNREG_HI
    WarpKernelFn lo_ch = nullptr, hi_ch = nullptr;  // shared-memory-cherry-only twins (CH = 1; nullptr: none)
    WarpKernelFn hi_gm = nullptr;                   // global-memory-cherry-only twin (CH = 2, 128 registers)
};

template <int E, bool GR, bool LS, bool W>
WarpKernel wk() {
    return WarpKernel{k_warp_engine<E, GR, LS, AD_WARP_MAXNREG, W>, k_warp_engine<E, GR, LS, AD_WARP_MAXNREG_HI, W>,
                      k_warp_engine<E, GR, LS, AD_WARP_MAXNREG, W, false, 1>,
                      k_warp_engine<E, GR, LS, AD_WARP_MAXNREG_HI, W, false, 1>,
                      k_warp_engine<E, GR, LS, AD_WARP_MAXNREG_HI, W, false, 2>};
}

// A14 instrumented LS kernels (ad_ls_params.phase_cycles): SIMT and TC engines
template <int E, bool W>
WarpKernel wk_instr() {
    return WarpKernel{k_warp_engine<E, true, true, AD_WARP_MAXNREG, W, true>,
                      k_warp_engine<E, true, true, AD_WARP_MAXNREG_HI, W, true>,
                      k_warp_engine<E, true, true, AD_WARP_MAXNREG, W, true, 1>,
                      k_warp_engine<E, true, true, AD_WARP_MAXNREG_HI, W, true, 1>,
                      k_warp_engine<E, true, true, AD_WARP_MAXNREG_HI, W, true, 2>};
}
WarpKernel pick_instr_kernel(int engine, bool wide) {
    if (engine == AD_ENGINE_TC) return wide ? wk_instr<1, true>() : wk_instr<1, false>();
    return wide ? wk_instr<0, true>() : wk_instr<0, false>();
}

template <bool W>
WarpKernel pick_warp_kernel_w(int engine, bool grad, bool ls) {
    if (ls) return engine == AD_ENGINE_TC        ? wk<1, true, true, W>()
                   : engine == AD_ENGINE_TC_FP16 ? wk<2, true, true, W>()
                                                 : wk<0, true, true, W>();
    if (!grad) return wk<0, false, false, W>();
    return engine == AD_ENGINE_TC ? wk<1, true, false, W>() : wk<0, true, false, W>();
}

// wide = some ligand the launch may touch has more than 32 genes
WarpKernel pick_warp_kernel(int engine, bool grad, bool ls, bool wide) {
    return wide ? pick_warp_kernel_w<true>(engine, grad, ls) : pick_warp_kernel_w<false>(engine, grad, ls);
}

// The ligands a pose_ligand launch may reference: the launch set, or every live ligand.
template <class F>
void for_each_launch_ligand(const ad_context* ctx, F f) {
    if (ctx->launch_set.empty()) {
        for (const LigSlot& o : ctx->ligs)
            if (o.live) f(o);
    } else {
        for (int id : ctx->launch_set)
            if (id < (int)ctx->ligs.size() && ctx->ligs[id].live) f(ctx->ligs[id]);
    }
}

bool launch_is_wide(const ad_context* ctx, ad_ligand_id lig, const int32_t* pose_ligand) {
    if (!pose_ligand) return 6 + ctx->ligs[lig].n_tors > 32;
    bool wide = false;
    for_each_launch_ligand(ctx, [&](const LigSlot& o) { wide |= 6 + o.n_tors > 32; });
    return wide;
}

int32_t common_checks(ad_context* ctx, ad_ligand_id lig, int32_t n_poses, const void* genes, int32_t stride) {
    if (!ctx) return fail(AD_ERR_INVALID_ARG, "ctx is NULL");
    if (!ctx->has_grid) return fail(AD_ERR_STATE, "no grid uploaded");
    if (lig < 0 || lig >= (int)ctx->ligs.size() || !ctx->ligs[lig].live) return fail(AD_ERR_INVALID_ARG, "bad ligand id %d", lig);
    if (n_poses < 0) return fail(AD_ERR_INVALID_ARG, "n_poses < 0");
    if (n_poses > 0 && !genes) return fail(AD_ERR_INVALID_ARG, "genes is NULL");
    if (stride < 6 + ctx->ligs[lig].n_tors) return fail(AD_ERR_INVALID_ARG, "geno_stride %d < 6 + n_tors", stride);
    return AD_OK;
}

// pose_ligand launches may touch any live ligand; the scoring constants are kernel
// parameters, so they must be identical across the live ligands
int32_t check_common_ff(ad_context* ctx, ad_ligand_id lig) {
    bool same = true;
    for_each_launch_ligand(ctx, [&](const LigSlot& o) { same &= memcmp(o.ff, ctx->ligs[lig].ff, sizeof(o.ff)) == 0; });
    if (!same)
        return fail(AD_ERR_INVALID_ARG, "pose_ligand launches need every referenced ligand uploaded with the same ad_ff_params");
    return AD_OK;
}

// Choose warps per CTA: the most resident warps per SM, ties -> fewer warps per CTA
// (finer load balance across SMs).
int32_t launch_warp(ad_context* ctx, LigSlot L, WarpKernel kern, KParams& p, int req_warps, cudaStream_t st,
                    bool tc_engine, int run_align = 8) {
    if (!tc_engine) L.scratch_bytes = L.scratch_simt;
    if (p.pose_ligand)  // any ligand of the launch set may be referenced: size for the largest footprint
        for_each_launch_ligand(ctx, [&](const LigSlot& o) {
            L.blob_bytes = std::max(L.blob_bytes, o.blob_bytes);
            L.scratch_bytes = std::max(L.scratch_bytes, tc_engine ? o.scratch_bytes : o.scratch_simt);
        });
    // Every pose costs the same.  A launch shape (register variant, W warps per CTA)
    // is scored by the modelled time of the busiest SM: it receives ceil(CTAs / SMs)
    // CTAs and runs them in waves of `blocks` resident CTAs; a wave of a warps
    // (a poses) takes a^(1 - gamma) time units, i.e. per-SM throughput grows as
    // a^gamma with the resident warps (partial latency hiding).  gamma = 0.48 fits
    // the measured config-2 shapes (tools/ab.py, ms per LS launch): W = 6 (4 CTAs =
    // 24 poses on the busiest SM) 4.14, W = 7 (3 CTAs = 21 poses) 3.87, W = 11
    // (22 poses) 3.87, W = 8 (24 poses) 4.02.  The 128-register twin executes
    // ~10 % fewer instructions and no spills: its time is scaled by 0.85 (config 3,
    // smem-bound at 16 warps/SM either way: 128.3 ms vs 147.7 ms for the 80-register
    // twin at 18).  Ties: less shared memory in use per SM (fewer blob copies: more L1
    // left for the grid gathers and spills), then more resident warps.
    // Mixed-ligand launches keep power-of-two CTA sizes (pose_ligand groups stay aligned).
    struct Cand { int w = 0, active = -1; double cost = 1e300; size_t sm_smem = 0; size_t smem = 0; WarpKernelFn k = nullptr; };
    Cand pick;
    static const int force = getenv("AD_MAXREG") ? atoi(getenv("AD_MAXREG")) : 0;  // A/B knob: 80 or 128
    // ligands with global-memory schedules (pre-decoded places of wide ligands, streamed
    // cherry records) run the 128-register kernels, which alone carry those loops
    // (config 3: 121.0 ms vs 130.6 ms on the 80-register kernels' record-decoding loop)
    bool pkg = L.pkg, ch = L.smem_cherry, gmc = L.gm_cherry;
    if (p.pose_ligand)
        for_each_launch_ligand(ctx, [&](const LigSlot& o) { pkg |= o.pkg; ch &= o.smem_cherry; gmc &= o.gm_cherry; });
    static const bool ch_on = !getenv("AD_NO_CH");  // A/B knob: generic kernels only
    if (ch && ch_on && kern.lo_ch) {  // every ligand of the launch runs shared-memory cherries: the cherry-only twins
        kern.lo = kern.lo_ch;
        kern.hi = kern.hi_ch;
    } else if (gmc && ch_on && kern.hi_gm) {  // ... global-memory cherries (128-register kernels only)
        kern.hi = kern.hi_gm;
    }
    // the decision depends on nothing else: cached (a config-1 score call is ~9 us of
    // kernel; the 64-candidate search must not add to it on every call)
    const ad_context::LaunchKey key{reinterpret_cast<const void*>(kern.lo), reinterpret_cast<const void*>(kern.hi),
                                    L.blob_bytes, L.scratch_bytes, p.n_poses, req_warps, p.pose_ligand ? 1 : 0,
                                    run_align, pkg ? 1 : 0};
    {
        std::lock_guard<std::mutex> lock(ctx->launch_mu);
        for (const auto& e : ctx->launch_cache)
            if (e.key == key) {
                p.smem_blob = L.blob_bytes;
                p.smem_scratch = L.scratch_bytes;
                const int grid = (p.n_poses + e.w - 1) / e.w;
                const WarpKernelFn k = reinterpret_cast<WarpKernelFn>(const_cast<void*>(e.k));
                k<<<grid, e.w * 32, e.smem, st>>>(p);
                ctx->last_maxreg = k == kern.hi ? AD_WARP_MAXNREG_HI : AD_WARP_MAXNREG;
                ctx->last_grid = grid;
                ctx->last_block = e.w * 32;
                ctx->last_smem = (int32_t)e.smem;
                CUDA_TRY(cudaGetLastError());
                return AD_OK;
            }
    }
    static const bool debug_launch = getenv("AD_DEBUG_LAUNCH") != nullptr;
    for (int v = 0; v < 2; ++v) {
        const WarpKernelFn k = v ? kern.hi : kern.lo;
        if (force && force != (v ? AD_WARP_MAXNREG_HI : AD_WARP_MAXNREG)) continue;
        if (pkg && !v) continue;
        for (int w = 1; w <= 32; ++w) {
            if (req_warps > 0 && w != req_warps) continue;
            // pose_ligand: CTA groups never straddle two ligands' poses -- powers of two
            // dividing the run alignment (ad.h: pop_per_run, else runs of 8)
            if (p.pose_ligand && ((w & (w - 1)) || run_align % w)) continue;
            const size_t smem = (size_t)L.blob_bytes + (size_t)w * L.scratch_bytes;
            if (smem > (size_t)ctx->max_smem_optin) continue;
            int blocks = 0;
            if (int32_t rc = occupancy(ctx, reinterpret_cast<const void*>(k), w * 32, smem, &blocks)) return rc;
            if (blocks <= 0) continue;
            const int active = blocks * w;
            const long ctas = (p.n_poses + w - 1) / w;
            const long per_sm = (ctas + ctx->n_sms - 1) / ctx->n_sms;  // CTAs on the busiest SM
            const long full = per_sm / blocks, rem = per_sm % blocks;
            const double g1 = 1.0 - 0.48;
            double cost = (double)full * std::pow((double)active, g1) + (rem ? std::pow((double)(rem * w), g1) : 0.0);
            if (v) cost *= 0.85;
            const size_t sm_smem = (size_t)std::min<long>(blocks, per_sm) * smem;  // in use on the busiest SM
            // shared memory in use is L1 taken from the grid gathers, the streamed records
            // and the spills: +10 % cost for a full SM (config 3, W = 2 / 4 / 8 / 16 -> 191 /
            // 159 / 143 / 135 KB per SM: 98.6 / 97.2 / 96.4 / 102.3 ms per LS launch; the
            // wave model alone picked W = 2)
            cost *= 1.0 + 0.1 * (double)sm_smem / (double)std::max(ctx->max_smem_optin, 1);
            if (debug_launch)
                fprintf(stderr, "[libad] regs=%d w=%d smem=%zu blocks/SM=%d active=%d ctas=%ld per_sm=%ld cost=%.3f\n",
                        v ? AD_WARP_MAXNREG_HI : AD_WARP_MAXNREG, w, smem, blocks, active, ctas, per_sm, cost);
            const bool better = cost < pick.cost - 1e-9 ||
                                (cost < pick.cost + 1e-9 && (sm_smem < pick.sm_smem || (sm_smem == pick.sm_smem && active > pick.active)));
            if (better) pick = Cand{w, active, cost, sm_smem, smem, k};
        }
    }
    const int best_w = pick.w, best_active = pick.active;
    const size_t best_smem = pick.smem;
    const WarpKernelFn best_k = pick.k;
    if (best_w == 0 || best_active <= 0)
        return fail(AD_ERR_LIMIT, "ligand footprint (%d B blob + %d B/warp) does not fit shared memory", L.blob_bytes,
                    L.scratch_bytes);
    p.smem_blob = L.blob_bytes;
    p.smem_scratch = L.scratch_bytes;
    {
        std::lock_guard<std::mutex> lock(ctx->launch_mu);
        if (ctx->launch_cache.size() < 4096)
            ctx->launch_cache.push_back({key, best_w, reinterpret_cast<const void*>(best_k), best_smem});
    }
    const int grid = (p.n_poses + best_w - 1) / best_w;
    best_k<<<grid, best_w * 32, best_smem, st>>>(p);
    ctx->last_maxreg = best_k == kern.hi ? AD_WARP_MAXNREG_HI : AD_WARP_MAXNREG;
    ctx->last_grid = grid;
    ctx->last_block = best_w * 32;
    ctx->last_smem = (int32_t)best_smem;
    CUDA_TRY(cudaGetLastError());
    return AD_OK;
}

KParams base_params(ad_context* ctx, ad_ligand_id lig, const int32_t* pose_ligand, int32_t n_poses, int32_t stride) {
    KParams p{};
    p.grid = ctx->grid;
    p.ligs = ctx->d_ligtab;
    p.lig = lig;
    p.pose_ligand = pose_ligand;
    p.n_poses = n_poses;
    p.stride = stride;
    p.err = ctx->d_err;
    p.err_seen = ctx->d_err_seen;
    p.n_ligs = (int32_t)ctx->ligs.size();
    p.max_iters = 1;
    p.pc = pair_const_from_ff(ctx->ligs[lig].ff);
    return p;
}

}  // namespace

extern "C" {

int32_t ad_score_poses(ad_context* ctx, ad_ligand_id lig, const int32_t* pose_ligand, int32_t n_poses,
                       const float* genes, int32_t geno_stride, float* energy, float* grad, float* aux,
                       void* stream) {
    NvtxRange nvtx_range("ad_score_poses");
    if (int32_t rc = common_checks(ctx, lig, n_poses, genes, geno_stride)) return rc;
    if (n_poses > 0 && !energy) return fail(AD_ERR_INVALID_ARG, "energy is NULL");
    if (pose_ligand) {
        if (int32_t rc = check_common_ff(ctx, lig)) return rc;
    }
    if (int32_t rc = set_device(ctx)) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    if (int32_t rc = check_device_err(ctx, st)) return rc;
    if (n_poses == 0) return AD_OK;
    KParams p = base_params(ctx, lig, pose_ligand, n_poses, geno_stride);
    p.genes = const_cast<float*>(genes);
    p.energy = energy;
    p.grad = grad;
    p.aux = aux;
    const bool want_grad = grad != nullptr || aux != nullptr;
    if (int32_t rc = launch_warp(ctx, ctx->ligs[lig],
                                 pick_warp_kernel(AD_ENGINE_SIMT, want_grad, false, launch_is_wide(ctx, lig, pose_ligand)),
                                 p, 0, st, false))
        return rc;
    return read_back_err(ctx, st);
}

int32_t ad_local_search(ad_context* ctx, ad_ligand_id lig, const int32_t* pose_ligand, int32_t n_poses, float* genes,
                        int32_t geno_stride, float* best_energy, float* run_best, int64_t* n_evals,
                        const ad_ls_params* prm, void* stream) {
    NvtxRange nvtx_range("ad_local_search");
    if (int32_t rc = common_checks(ctx, lig, n_poses, genes, geno_stride)) return rc;
    if (!prm) return fail(AD_ERR_INVALID_ARG, "params is NULL");
    if (prm->max_iters < 1) return fail(AD_ERR_INVALID_ARG, "max_iters must be >= 1");
    if (prm->engine < 0 || prm->engine > 4) return fail(AD_ERR_INVALID_ARG, "unknown engine %d", prm->engine);
    if (!(prm->rho >= 0.f && prm->rho < 1.f) || !(prm->eps > 0.f)) return fail(AD_ERR_INVALID_ARG, "need 0 <= rho < 1, eps > 0");
    if (n_poses > 0 && !best_energy) return fail(AD_ERR_INVALID_ARG, "best_energy is NULL");
    if (pose_ligand) {
        if (int32_t rc = check_common_ff(ctx, lig)) return rc;
    }
    if (run_best && (prm->pop_per_run <= 0 || n_poses % prm->pop_per_run))
        return fail(AD_ERR_INVALID_ARG, "run_best needs pop_per_run > 0 dividing n_poses");
    if (int32_t rc = set_device(ctx)) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    if (int32_t rc = check_device_err(ctx, st)) return rc;
    if (n_poses == 0) return AD_OK;
    KParams p = base_params(ctx, lig, pose_ligand, n_poses, geno_stride);
    p.genes = genes;
    p.energy = best_energy;
    p.trace = prm->trace;
    p.n_evals = n_evals;
    p.max_iters = prm->max_iters;
    p.rho = prm->rho;
    p.eps = prm->eps;
    p.phase_cycles = prm->phase_cycles;
    if (p.phase_cycles && prm->engine == AD_ENGINE_TC_FP16)
        return fail(AD_ERR_INVALID_ARG, "phase_cycles: no instrumented build of the TC_FP16 engine");
    const LigSlot& L = ctx->ligs[lig];
    if (prm->engine == AD_ENGINE_PAPER_BASELINE || prm->engine == AD_ENGINE_PAPER_TCEC) {
        const bool tcec = prm->engine == AD_ENGINE_PAPER_TCEC;
        int threads = prm->warps_per_cta > 0 ? prm->warps_per_cta : 64;
        if (threads % 32 || threads < 32 || threads > 256) return fail(AD_ERR_INVALID_ARG, "baseline block size %d", threads);
        if (6 + L.n_tors > threads) return fail(AD_ERR_INVALID_ARG, "baseline needs >= 6 + n_tors threads");
        int32_t blob = L.base_bytes, bscr = block_scratch_layout(L.n_atoms, L.n_tors, tcec ? threads : 0).bytes;
        if (pose_ligand)
            for_each_launch_ligand(ctx, [&](const LigSlot& o) {
                blob = std::max(blob, o.base_bytes);
                bscr = std::max(bscr, block_scratch_layout(o.n_atoms, o.n_tors, tcec ? threads : 0).bytes);
            });
        const size_t smem = (size_t)blob + bscr;
        if (smem > (size_t)ctx->max_smem_optin) return fail(AD_ERR_LIMIT, "ligand too large for the baseline engine");
        void (*kern)(const KParams) = p.phase_cycles ? (tcec ? k_block_baseline<true, true> : k_block_baseline<false, true>)
                                                     : (tcec ? k_block_baseline<true> : k_block_baseline<false>);
        if (int32_t rc = opt_in_smem(ctx, reinterpret_cast<const void*>(kern))) return rc;
        p.smem_blob = blob;
        p.smem_scratch = bscr;
        kern<<<n_poses, threads, smem, st>>>(p);
        ctx->last_grid = n_poses;
        ctx->last_block = threads;
        ctx->last_smem = (int32_t)smem;
        CUDA_TRY(cudaGetLastError());
    } else {
        int w = prm->warps_per_cta;
        if (w < 0 || w > 32) return fail(AD_ERR_INVALID_ARG, "warps_per_cta %d not in 0..32", w);
        const bool wide = launch_is_wide(ctx, lig, pose_ligand);
        const WarpKernel k = p.phase_cycles ? pick_instr_kernel(prm->engine, wide)
                                            : pick_warp_kernel(prm->engine, true, true, wide);
        // with pose_ligand and pop_per_run > 0, a ligand's poses come in whole runs
        int align = 8;
        if (pose_ligand && prm->pop_per_run > 0) {
            align = 1;
            while (align < 8 && prm->pop_per_run % (2 * align) == 0) align *= 2;
        }
        if (pose_ligand && w > 0 && ((w & (w - 1)) || align % w))
            return fail(AD_ERR_INVALID_ARG, "pose_ligand launch: warps_per_cta %d must be a power of two dividing %d", w,
                        align);
        if (int32_t rc = launch_warp(ctx, L, k, p, w, st, prm->engine == AD_ENGINE_TC || prm->engine == AD_ENGINE_TC_FP16,
                                     align))
            return rc;
    }
    if (run_best) {
        const int runs = n_poses / prm->pop_per_run;
        // the whole genotype row is copied: with pose_ligand the runs of one call
        // belong to ligands with different gene counts
        k_best_of_run<<<(runs + 3) / 4, 128, 0, st>>>(best_energy, genes, geno_stride,
                                                      pose_ligand ? geno_stride : 6 + L.n_tors, prm->pop_per_run,
                                                      runs, run_best);
        CUDA_TRY(cudaGetLastError());
    }
    return read_back_err(ctx, st);
}

int32_t ad_lga_run(ad_context* ctx, ad_ligand_id lig, int32_t n_runs, float* genes, int32_t geno_stride,
                   float* energies, float* run_best, int64_t* n_evals, int32_t* n_gens, const ad_lga_params* prm,
                   void* stream) {
    NvtxRange nvtx_range("ad_lga_run");
    if (!prm) return fail(AD_ERR_INVALID_ARG, "params is NULL");
    const int pop = prm->pop_size;
    if (n_runs < 0 || pop < 2 || pop > 4096) return fail(AD_ERR_INVALID_ARG, "need n_runs >= 0, 2 <= pop_size <= 4096");
    const int64_t n_ind64 = (int64_t)n_runs * pop;
    if (n_ind64 > (1 << 30)) return fail(AD_ERR_LIMIT, "population too large");
    const int n_ind = (int)n_ind64;
    if (int32_t rc = common_checks(ctx, lig, n_ind, genes, geno_stride)) return rc;
    if (n_ind > 0 && !energies) return fail(AD_ERR_INVALID_ARG, "energies is NULL");
    const ad_ls_params& ls = prm->ls;
    if (ls.engine != AD_ENGINE_SIMT && ls.engine != AD_ENGINE_TC && ls.engine != AD_ENGINE_TC_FP16)
        return fail(AD_ERR_INVALID_ARG, "LGA runs the warp engines (SIMT, TC, TC_FP16)");
    if (ls.max_iters < 1 || !(ls.rho >= 0.f && ls.rho < 1.f) || !(ls.eps > 0.f))
        return fail(AD_ERR_INVALID_ARG, "bad LS parameters");
    if (ls.warps_per_cta < 0 || ls.warps_per_cta > 32) return fail(AD_ERR_INVALID_ARG, "warps_per_cta not in 0..32");
    if (prm->elitism < 0 || prm->elitism > pop || prm->max_gens < 0 || prm->max_evals < 0)
        return fail(AD_ERR_INVALID_ARG, "bad GA parameters");
    if (int32_t rc = set_device(ctx)) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    if (int32_t rc = check_device_err(ctx, st)) return rc;
    if (n_ind == 0) return AD_OK;
    const LigSlot& L = ctx->ligs[lig];
    const int S = geno_stride;
    GaParams G{pop, 6 + L.n_tors, S, prm->elitism, prm->cross_rate, prm->mut_rate, prm->tour_rate, prm->ls_rate,
               prm->dmov, prm->dang, prm->seed};
    // scratch: next population, LS list + genes + energies, per-run counters
    float *d_next = nullptr, *d_lsg = nullptr, *d_lse = nullptr;
    int32_t *d_list = nullptr, *d_cnt = nullptr, *d_per = nullptr, *d_done = nullptr, *d_gens = nullptr,
            *d_ndone = nullptr;
    int64_t* d_evals = nullptr;
    auto cleanup = [&]() {
        cudaFree(d_next); cudaFree(d_lsg); cudaFree(d_lse); cudaFree(d_list); cudaFree(d_cnt);
        cudaFree(d_per); cudaFree(d_done); cudaFree(d_gens); cudaFree(d_ndone); cudaFree(d_evals);
    };
#define LGA_TRY(expr)                                                                     \
    do {                                                                                  \
        cudaError_t e_ = (expr);                                                          \
        if (e_ != cudaSuccess) {                                                          \
            cleanup();                                                                    \
            return fail(e_ == cudaErrorMemoryAllocation ? AD_ERR_OOM : AD_ERR_CUDA, "%s: %s", #expr, \
                        cudaGetErrorString(e_));                                          \
        }                                                                                 \
    } while (0)
    const size_t rows = (size_t)n_ind * S * sizeof(float);
    LGA_TRY(cudaMalloc(&d_next, rows));
    LGA_TRY(cudaMalloc(&d_lsg, rows));
    LGA_TRY(cudaMalloc(&d_lse, sizeof(float) * n_ind));
    LGA_TRY(cudaMalloc(&d_list, sizeof(int32_t) * n_ind));
    LGA_TRY(cudaMalloc(&d_cnt, sizeof(int32_t)));
    LGA_TRY(cudaMalloc(&d_per, sizeof(int32_t) * n_runs));
    LGA_TRY(cudaMalloc(&d_done, sizeof(int32_t) * n_runs));
    LGA_TRY(cudaMalloc(&d_gens, sizeof(int32_t) * n_runs));
    LGA_TRY(cudaMalloc(&d_ndone, sizeof(int32_t)));
    LGA_TRY(cudaMalloc(&d_evals, sizeof(int64_t) * n_runs));
    LGA_TRY(cudaMemsetAsync(d_cnt, 0, sizeof(int32_t), st));
    LGA_TRY(cudaMemsetAsync(d_per, 0, sizeof(int32_t) * n_runs, st));
    LGA_TRY(cudaMemsetAsync(d_done, 0, sizeof(int32_t) * n_runs, st));
    LGA_TRY(cudaMemsetAsync(d_gens, 0, sizeof(int32_t) * n_runs, st));
    LGA_TRY(cudaMemsetAsync(d_ndone, 0, sizeof(int32_t), st));
    // evaluations of the initial population: pop per run
    {
        std::vector<int64_t> e0(n_runs, (int64_t)pop);
        LGA_TRY(cudaMemcpyAsync(d_evals, e0.data(), sizeof(int64_t) * n_runs, cudaMemcpyHostToDevice, st));
        LGA_TRY(cudaStreamSynchronize(st));
    }
    auto score_all = [&](float* g) -> int32_t {
        KParams p = base_params(ctx, lig, nullptr, n_ind, S);
        p.genes = g;
        p.energy = energies;
        return launch_warp(ctx, L, pick_warp_kernel(AD_ENGINE_SIMT, false, false, launch_is_wide(ctx, lig, nullptr)), p, 0, st, false);
    };
    if (int32_t rc = score_all(genes)) { cleanup(); return rc; }
    KParams lp = base_params(ctx, lig, nullptr, n_ind, S);
    lp.genes = d_lsg;
    lp.energy = d_lse;
    lp.max_iters = ls.max_iters;
    lp.rho = ls.rho;
    lp.eps = ls.eps;
    lp.n_active = d_cnt;
    const bool tc = ls.engine != AD_ENGINE_SIMT;
    WarpKernel ls_kern = pick_warp_kernel(ls.engine, true, true, launch_is_wide(ctx, lig, nullptr));
    // a run that starts finished (budget already spent) takes no generation
    const bool start_done = prm->max_gens == 0 || (int64_t)pop >= prm->max_evals;
    int gen = 0;
    if (start_done) {
        std::vector<int32_t> ones(n_runs, 1);
        LGA_TRY(cudaMemcpyAsync(d_done, ones.data(), sizeof(int32_t) * n_runs, cudaMemcpyHostToDevice, st));
        LGA_TRY(cudaStreamSynchronize(st));
    }
    float* cur = genes;
    float* nxt = d_next;
    for (; !start_done; ++gen) {
        // GA(population) -> scores of the new individuals
        k_ga_generation<<<n_runs, 128, pop, st>>>(G, cur, energies, nxt, d_done, (uint32_t)gen);
        LGA_TRY(cudaGetLastError());
        std::swap(cur, nxt);
        if (int32_t rc = score_all(cur)) { cleanup(); return rc; }
        // LS(population): compacted list, gather, ADADELTA, scatter back (Lamarckian)
        k_ga_ls_select<<<n_runs, 128, 0, st>>>(G, d_done, (uint32_t)gen, d_list, d_cnt, d_per);
        LGA_TRY(cudaGetLastError());
        // the LS launch is shaped for the individuals actually selected (ls_rate of the
        // population): read back the count first, so the CTAs spread over every SM instead
        // of a grid sized for the whole population whose tail CTAs exit at once (config 2,
        // ls_rate 0.8: ~2400 of 3000 poses on ~113 of 148 SMs)
        int32_t h_cnt = 0;
        LGA_TRY(cudaMemcpyAsync(&h_cnt, d_cnt, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        const int rb = std::min(65535, (n_ind * S + 255) / 256);
        k_ga_rows<<<rb, 256, 0, st>>>(d_list, d_cnt, S, cur, d_lsg, false, nullptr, nullptr);
        LGA_TRY(cudaGetLastError());
        LGA_TRY(cudaStreamSynchronize(st));
        lp.n_poses = std::min(std::max(h_cnt, 0), n_ind);
        if (lp.n_poses > 0)
            if (int32_t rc = launch_warp(ctx, L, ls_kern, lp, ls.warps_per_cta, st, tc)) { cleanup(); return rc; }
        k_ga_rows<<<rb, 256, 0, st>>>(d_list, d_cnt, S, d_lsg, cur, true, d_lse, energies);
        LGA_TRY(cudaGetLastError());
        k_ga_update<<<(n_runs + 127) / 128, 128, 0, st>>>(n_runs, pop, ls.max_iters, prm->max_evals, prm->max_gens,
                                                         d_done, d_evals, d_gens, d_per, d_cnt, d_ndone);
        LGA_TRY(cudaGetLastError());
        int32_t h_done = 0;
        LGA_TRY(cudaMemcpyAsync(&h_done, d_ndone, sizeof(int32_t), cudaMemcpyDeviceToHost, st));
        LGA_TRY(cudaStreamSynchronize(st));
        if (h_done >= n_runs) break;
    }
    if (cur != genes) LGA_TRY(cudaMemcpyAsync(genes, cur, rows, cudaMemcpyDeviceToDevice, st));
    if (run_best) {
        k_best_of_run<<<(n_runs + 3) / 4, 128, 0, st>>>(energies, genes, S, G.n_genes, pop, n_runs, run_best);
        LGA_TRY(cudaGetLastError());
    }
    if (n_evals) LGA_TRY(cudaMemcpyAsync(n_evals, d_evals, sizeof(int64_t) * n_runs, cudaMemcpyDeviceToDevice, st));
    if (n_gens) LGA_TRY(cudaMemcpyAsync(n_gens, d_gens, sizeof(int32_t) * n_runs, cudaMemcpyDeviceToDevice, st));
    LGA_TRY(cudaStreamSynchronize(st));
#undef LGA_TRY
    cleanup();
    return read_back_err(ctx, st);
}

int32_t ad_reduce_blocks(ad_context* ctx, int32_t engine, int32_t n_blocks, int32_t n_partials, int32_t n_comp,
                         const float* partials, float* out, void* stream) {
    NvtxRange nvtx_range("ad_reduce_blocks");
    if (!ctx || !partials || !out) return fail(AD_ERR_INVALID_ARG, "null argument");
    if (n_blocks < 0) return fail(AD_ERR_INVALID_ARG, "n_blocks < 0");
    if (n_partials < 32 || n_partials > 1024 || n_partials % 32) return fail(AD_ERR_INVALID_ARG, "n_partials %d", n_partials);
    if (n_comp < 1 || n_comp > 64) return fail(AD_ERR_INVALID_ARG, "n_comp %d not in [1,64]", n_comp);
    if (int32_t rc = set_device(ctx)) return rc;
    if (n_blocks == 0) return AD_OK;
    cudaStream_t st = (cudaStream_t)stream;
    const int nw = n_partials / 32;
    if (engine == AD_ENGINE_SIMT) {
        const int cmax = n_comp <= 8 ? 8 : n_comp <= 16 ? 16 : n_comp <= 32 ? 32 : 64;
        const size_t smem = sizeof(float) * nw * cmax;
        switch (cmax) {
            case 8: k_reduce_simt<8><<<n_blocks, n_partials, smem, st>>>(partials, out, n_comp); break;
            case 16: k_reduce_simt<16><<<n_blocks, n_partials, smem, st>>>(partials, out, n_comp); break;
            case 32: k_reduce_simt<32><<<n_blocks, n_partials, smem, st>>>(partials, out, n_comp); break;
            default: k_reduce_simt<64><<<n_blocks, n_partials, smem, st>>>(partials, out, n_comp); break;
        }
    } else if (engine == AD_ENGINE_TC) {
        const int c8 = (n_comp + 7) & ~7;
        const size_t smem = sizeof(float) * ((size_t)nw * 32 * c8 + (size_t)nw * c8);
        if (smem > (size_t)ctx->max_smem_optin) return fail(AD_ERR_LIMIT, "TC reduce staging too large");
        CUDA_TRY(cudaFuncSetAttribute(k_reduce_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        k_reduce_tc<<<n_blocks, n_partials, smem, st>>>(partials, out, n_comp);
    } else if (engine == AD_ENGINE_TC_FP16) {
        const int c8 = (n_comp + 7) & ~7;
        const size_t smem = sizeof(float) * (size_t)nw * 32 * c8 + sizeof(uint16_t) * (size_t)nw * c8;
        if (smem > (size_t)ctx->max_smem_optin) return fail(AD_ERR_LIMIT, "TC reduce staging too large");
        CUDA_TRY(cudaFuncSetAttribute(k_reduce_tc_fp16, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
        k_reduce_tc_fp16<<<n_blocks, n_partials, smem, st>>>(partials, out, n_comp);
    } else if (engine == AD_ENGINE_PAPER_BASELINE) {
        k_reduce_paper<<<n_blocks, n_partials, 0, st>>>(partials, out, n_comp);
    } else {
        return fail(AD_ERR_INVALID_ARG, "unknown engine %d", engine);
    }
    CUDA_TRY(cudaGetLastError());
    return AD_OK;
}

// Host-only inspection hook (not part of include/ad.h; no GPU needed): run the
// intra-pair scheduler on a pair list of atoms 0..n_atoms-1.  Writes the number of
// steps and slots; copies up to `cap` records (64 per step) to out_rec.
int32_t adx_debug_schedule(int32_t n_atoms, int32_t n_pairs, const int32_t* pairs, int32_t* out_steps,
                           int32_t* out_slots, uint32_t* out_rec, int32_t cap, int32_t* out_atom_slot) {
    if (n_atoms < 1 || n_atoms > AD_MAX_ATOMS || n_pairs < 0 || (n_pairs && !pairs) || !out_steps || !out_slots)
        return fail(AD_ERR_INVALID_ARG, "bad arguments");
    std::vector<int> pi(n_pairs), pj(n_pairs), ptp(n_pairs, 0);
    std::vector<float> pd(n_pairs, 0.f);
    for (int q = 0; q < n_pairs; ++q) {
        pi[q] = pairs[2 * q];
        pj[q] = pairs[2 * q + 1];
        if (pi[q] < 0 || pi[q] >= n_atoms || pj[q] < 0 || pj[q] >= n_atoms || pi[q] == pj[q])
            return fail(AD_ERR_INVALID_ARG, "bad pair %d", q);
    }
    const std::vector<int> slot = balance_slots(n_atoms, pi, pj);
    for (int q = 0; q < n_pairs; ++q) {
        pi[q] = slot[pi[q]];
        pj[q] = slot[pj[q]];
    }
    if (out_atom_slot)
        for (int a = 0; a < n_atoms; ++a) out_atom_slot[a] = slot[a];
    const Schedule s = schedule_pairs(n_atoms, pi, pj, ptp, pd, pd);
    *out_steps = s.rounds;
    *out_slots = s.slots;
    if (out_rec)
        for (int q = 0; q < std::min<int>(cap, (int)s.rec.size()); ++q) out_rec[q] = s.rec[q];
    return AD_OK;
}

// Host-only inspection hook (not part of include/ad.h; no GPU needed): the cherry
// schedule of a pair list (storage rows from balance_slots, as at upload).  out
// receives [steps*32][8] int32: centre, end0, end1 (rows), pair0, pair1 (ids),
// slot of centre / end0 / end1 (-1 = empty).
int32_t adx_debug_cherries(int32_t n_atoms, int32_t n_pairs, const int32_t* pairs, int32_t effort, int32_t* out_steps,
                           int32_t* out_slots, int32_t* out, int32_t cap_lanes, int32_t* out_atom_slot) {
    if (n_atoms < 1 || n_atoms > AD_MAX_ATOMS || n_pairs < 0 || (n_pairs && !pairs) || !out_steps || !out_slots)
        return fail(AD_ERR_INVALID_ARG, "bad arguments");
    std::vector<int> pi(n_pairs), pj(n_pairs);
    for (int q = 0; q < n_pairs; ++q) {
        pi[q] = pairs[2 * q];
        pj[q] = pairs[2 * q + 1];
        if (pi[q] < 0 || pi[q] >= n_atoms || pj[q] < 0 || pj[q] >= n_atoms || pi[q] == pj[q])
            return fail(AD_ERR_INVALID_ARG, "bad pair %d", q);
    }
    const std::vector<int> slot = balance_slots(n_atoms, pi, pj);
    for (int q = 0; q < n_pairs; ++q) {
        pi[q] = slot[pi[q]];
        pj[q] = slot[pj[q]];
    }
    if (out_atom_slot)
        for (int a = 0; a < n_atoms; ++a) out_atom_slot[a] = slot[a];
    const CherrySchedule S = schedule_cherries(npad_of(n_atoms), pi, pj, effort, 1 << 30, cherry_max_slots(npad_of(n_atoms)));
    *out_steps = S.steps;
    *out_slots = S.slots;
    if (out)
        for (int q = 0; q < std::min<int>(cap_lanes, (int)S.lane.size()); ++q) {
            const CherryLane& L = S.lane[q];
            const int v[8] = {L.c, L.e[0], L.e[1], L.p[0], L.p[1], L.kc, L.ke[0], L.ke[1]};
            for (int k = 0; k < 8; ++k) out[8 * q + k] = v[k];
        }
    return AD_OK;
}

// Host-only inspection hook (not in include/ad.h): the pair loop a ligand runs --
// 1 shared-memory cherries (the CH = 1 kernels), 2 global-memory cherries (CH = 2),
// 0 any other (generic kernels), -1 bad id.  Launch buckets of one kind run the twins.
int32_t adx_pair_loop(ad_context* ctx, int32_t lig) {
    if (!ctx || lig < 0 || lig >= (int)ctx->ligs.size() || !ctx->ligs[lig].live) return -1;
    const LigSlot& L = ctx->ligs[lig];
    return L.smem_cherry ? 1 : L.gm_cherry ? 2 : 0;
}

// Host-only inspection hook (not in include/ad.h): register budget of the last
// warp-engine launch (AD_WARP_MAXNREG or AD_WARP_MAXNREG_HI).
int32_t adx_last_maxreg(ad_context* ctx) { return ctx ? ctx->last_maxreg : 0; }

int32_t ad_last_launch(ad_context* ctx, int32_t* grid, int32_t* block, int32_t* smem_bytes) {
    if (!ctx) return fail(AD_ERR_INVALID_ARG, "ctx is NULL");
    if (grid) *grid = ctx->last_grid;
    if (block) *block = ctx->last_block;
    if (smem_bytes) *smem_bytes = ctx->last_smem;
    return AD_OK;
}

int32_t ad_sync(ad_context* ctx, void* stream) {
    if (!ctx) return fail(AD_ERR_INVALID_ARG, "ctx is NULL");
    if (int32_t rc = set_device(ctx)) return rc;
    cudaStream_t st = (cudaStream_t)stream;
    CUDA_TRY(cudaStreamSynchronize(st));
    int32_t h = 0;
    CUDA_TRY(cudaMemcpy(&h, ctx->d_err, sizeof(int32_t), cudaMemcpyDeviceToHost));
    ctx->err_pending = false;
    *reinterpret_cast<volatile int32_t*>(ctx->h_err) = 0;
    if (h) {
        CUDA_TRY(cudaMemset(ctx->d_err, 0, sizeof(int32_t)));
        return report_device_err(h);
    }
    return AD_OK;
}

int32_t ad_query(ad_context* ctx, ad_ligand_id lig, int32_t* n_sms, int32_t* smem_per_pose, int32_t* blob_bytes) {
    if (!ctx) return fail(AD_ERR_INVALID_ARG, "ctx is NULL");
    if (n_sms) *n_sms = ctx->n_sms;
    if (lig >= 0) {
        if (lig >= (int)ctx->ligs.size() || !ctx->ligs[lig].live) return fail(AD_ERR_INVALID_ARG, "bad ligand id %d", lig);
        if (smem_per_pose) *smem_per_pose = ctx->ligs[lig].scratch_bytes;
        if (blob_bytes) *blob_bytes = ctx->ligs[lig].blob_bytes;
    }
    return AD_OK;
}

}  // extern "C"
