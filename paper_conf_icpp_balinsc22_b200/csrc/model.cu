// model.cu — executor of the MG-GCN hot path on B200: buffer plan (§4.2,
// P:827-901), staged SpMM with double-buffered broadcast (§4.1 P:705-720,
// §4.3), per-layer order choice (§4.4), loss, backward
// (Eq. 8-11), W_G reduction and Adam.
//
// Streams: stream 0 = compute, stream 1 = communication.
// Communication is NCCL (one process per GPU, nlocal = 1) or, for testing
// the P-stage pipeline on one GPU, LOOPBACK (all P ranks in this model,
// broadcasts = device copies on the comm stream with the same event graph).
#include <nccl.h>
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <chrono>
#include <thread>
#include <cmath>
#include <cstring>
#include <new>
#include <string>
#include <tuple>
#include <vector>

#include "internal.h"
#include "kernels.cuh"

using namespace mggcn;

namespace {

enum Order { G_ORDER = 0, S_ORDER = 1 };   // GeMM-first / SpMM-first (§4.4)
enum State { ST_READY = 0, ST_FWD = 1, ST_BWD = 2 };
// PC_DENSE: the dense-block kernels of an SpMM stage, recorded inside (and counted in) its PC_SPMM scope
enum ProfClass { PC_SPMM = 0, PC_GEMM, PC_LOSS, PC_ADAM, PC_BCAST, PC_ALLRED, PC_OTHER, PC_DENSE, PC_N };

struct Bump {
    char* base = nullptr;
    size_t off = 0;
    template <typename T>
    T* take(size_t count) {
        off = (off + 255) & ~size_t(255);
        T* p = base ? reinterpret_cast<T*>(base + off) : nullptr;
        off += sizeof(T) * (count ? count : 1);
        return p;
    }
};

struct HostItems {
    std::vector<int4> items, splits;
    int64_t nslots = 0;
    int64_t n_nonempty = 0;   // items[0, n_nonempty): hub segments and non-empty rows; then empty rows
    int64_t split = kSplit;   // segment length used for this tile
};

// Work items of one tile: hub rows (> kSplit entries) are cut into segments
// (first, so the long work starts early); every other row is one item, in
// `order` (the rows sorted by ORIGINAL vertex id: neighbouring original ids
// share neighbourhoods in the skewed input order, so warps of one SM that run
// consecutive items reuse gathered rows in L1/L2; numbering is unchanged).
void build_items(const HostTile& t, HostItems& h, const std::vector<int32_t>& order) {
    const auto& rp = t.rowptr;
    static int split_env = -1;
    if (split_env < 0) {
        const char* e = getenv("MGGCN_SPMM_SPLIT");
        split_env = e ? atoi(e) : 0;
        if (split_env != 0 && (split_env < 32 || split_env > 65536)) split_env = 0;
    }
    const int64_t kSplit = split_env ? split_env : split_for(rp.back());
    for (int64_t r = 0; r < t.nrows; ++r) {
        const int64_t len = rp[r + 1] - rp[r];
        if (len > kSplit) {
            const int64_t nseg = (len + kSplit - 1) / kSplit;
            h.splits.push_back(make_int4((int)r, (int)h.nslots, (int)nseg, 0));
            for (int64_t s = 0; s < nseg; ++s) {
                const int64_t b = rp[r] + s * kSplit, e = std::min<int64_t>(rp[r + 1], b + kSplit);
                h.items.push_back(make_int4((int)r, (int)b, (int)e, (int)(h.nslots + s)));
            }
            h.nslots += nseg;
        }
    }
    h.split = kSplit;
    // Empty rows go last: an accumulating middle stage skips them (adding an empty row's zero
    // sum is a no-op), which saves their output read-modify-write (SpmmTile::n_items_nz).
    for (int32_t r : order) {
        const int64_t len = rp[r + 1] - rp[r];
        if (len > 0 && len <= kSplit) h.items.push_back(make_int4(r, rp[r], rp[r + 1], -1));
    }
    h.n_nonempty = (int64_t)h.items.size();
    for (int32_t r : order)
        if (rp[r + 1] == rp[r]) h.items.push_back(make_int4(r, rp[r], rp[r + 1], -1));
}

// Duplicate entries (multi-edges, reading C19) are adjacent within a row
// (tiles are sorted by column); merge them: value = multiplicity for a
// pattern-only graph (Â_uv = mult / deg(v)), else the fp32 sum of the Â values.
void coalesce(const HostTile& t, HostTile& o) {
    o.nrows = t.nrows;
    o.ncols = t.ncols;
    o.col0 = t.col0;
    o.rowptr.assign(t.nrows + 1, 0);
    o.col.clear();
    o.val.clear();
    o.col.reserve(t.col.size());
    o.val.reserve(t.col.size());
    const bool pat = t.val.empty();
    for (int64_t r = 0; r < t.nrows; ++r) {
        const int64_t b = t.rowptr[r], e = t.rowptr[r + 1];
        const size_t start = o.col.size();
        for (int64_t q = b; q < e; ++q) {
            const float v = pat ? 1.0f : t.val[q];
            if (o.col.size() > start && o.col.back() == t.col[q]) o.val.back() += v;
            else {
                o.col.push_back(t.col[q]);
                o.val.push_back(v);
            }
        }
        o.rowptr[r + 1] = (int32_t)o.col.size();
    }
}

// L2 priority classes of a tile's columns (SpmmTile::hot_enc): the columns are
// ranked by reuse (entries per column, descending; ties by column id) and the
// device copy of the index carries hot_class_of(rank) in bits 24..31.  Used
// only for blocks whose 128-float slice exceeds the L2 (R-MAT hubs are reused
// across the whole tile; the rest of the block streams through).
bool want_hot_classes(const HostTile& ht) {
    static int env = -1;
    static int64_t l2 = 0;
    if (env < 0) {
        const char* e = getenv("MGGCN_SPMM_HOTCLS");
        env = e ? atoi(e) : 0;   // opt-in: no gain on Products-shaped blocks (profiles/r01_hot_sweep.log)
        int dev = 0, v = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&v, cudaDevAttrL2CacheSize, dev);
        l2 = v;
    }
    if (env == 0 || ht.ncols > ((int64_t)1 << 24)) return false;
    return env == 2 || (l2 > 0 && ht.ncols * 512 > l2);   // 2: always (tests)
}

std::vector<int32_t> encode_hot_classes(const HostTile& ht) {
    std::vector<int64_t> cnt(ht.ncols, 0);
    for (int32_t c : ht.col) ++cnt[c];
    std::vector<int32_t> ord(ht.ncols);
    for (int64_t c = 0; c < ht.ncols; ++c) ord[c] = (int32_t)c;
    std::stable_sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) { return cnt[a] > cnt[b]; });
    std::vector<uint32_t> cls(ht.ncols);
    for (int64_t r = 0; r < ht.ncols; ++r) cls[ord[r]] = (uint32_t)std::min(255, hot_class_of(r));
    std::vector<int32_t> out(ht.col.size());
    for (size_t e = 0; e < ht.col.size(); ++e) out[e] = (int32_t)((cls[ht.col[e]] << 24) | (uint32_t)ht.col[e]);
    return out;
}

// Stage groups: the tile of a group is the row-wise concatenation of the
// group's S column tiles, tile t's local column c becoming t * stride + c
// (stride = max_j n_j, the BC slot pitch in rows).  Entries of a row stay in
// (block, column) order; values are kept if any tile has them.
void merge_group_tiles(const std::vector<const HostTile*>& tiles, int64_t stride, HostTile& o) {
    const int64_t S = (int64_t)tiles.size();
    o.nrows = tiles[0]->nrows;
    o.ncols = S * stride;
    o.col0 = 0;
    bool vals = false;
    size_t nnz = 0;
    for (const HostTile* t : tiles) {
        vals = vals || !t->val.empty();
        nnz += t->col.size();
    }
    o.rowptr.assign(o.nrows + 1, 0);
    o.col.clear();
    o.val.clear();
    o.col.reserve(nnz);
    if (vals) o.val.reserve(nnz);
    for (int64_t r = 0; r < o.nrows; ++r) {
        for (int64_t t = 0; t < S; ++t) {
            const HostTile& h = *tiles[t];
            for (int32_t e = h.rowptr[r]; e < h.rowptr[r + 1]; ++e) {
                o.col.push_back((int32_t)(t * stride + h.col[e]));
                if (vals) o.val.push_back(h.val.empty() ? 1.0f : h.val[e]);
            }
        }
        o.rowptr[r + 1] = (int32_t)o.col.size();
    }
}

struct Rank {
    const mggcn_part_s* part = nullptr;
    int rank = 0;
    int rep = 0;                     // replica index (MGGCN_F_REPL2: rank (i, r) = r * P' + i)
    int64_t rows = 0, row_off = 0;   // row_off: offset inside the model's local rows
    std::vector<SpmmTile> F, B;
    std::vector<HostItems> hF, hB;
    // the tiles as uploaded: the partition's tiles, or (default) a copy with
    // duplicate entries coalesced into one entry whose value is the
    // multiplicity (pattern-only) or the sum of the values (weighted)
    std::vector<HostTile> cF, cB;
    bool coalesced = false;
    const HostTile& tF(int j) const { return coalesced ? cF[j] : part->F[j]; }
    const HostTile& tB(int j) const {
        if (coalesced) return part->shared_fb ? cF[j] : cB[j];
        return part->tileB(j);
    }
    // dense blocks of the launched tiles (plan_dense; DESIGN §6 "Dense blocks"): when active,
    // the launch tile is the residual CSR and the blocks run on the tensor cores
    std::vector<DenseHost> dF, dB, dgF, dgB;
    const HostTile& lF(int j) const { return (j < (int)dF.size() && dF[j].active) ? dF[j].resid : tF(j); }
    const HostTile& lB(int j) const {
        if (part->shared_fb) return lF(j);
        return (j < (int)dB.size() && dB[j].active) ? dB[j].resid : tB(j);
    }
    const HostTile& lgF(int g) const { return (g < (int)dgF.size() && dgF[g].active) ? dgF[g].resid : gF[g]; }
    const HostTile& lgB(int g) const { return (g < (int)dgB.size() && dgB[g].active) ? dgB[g].resid : gB[g]; }
    uint8_t* dense_bimg = nullptr;   // B-image scratch shared by the tiles' dense launches
    float* dense_partial = nullptr;  // partial products of split row groups (same sharing)
    float* inv_deg = nullptr;
    float* Xs = nullptr;             // current input buffer (= Xbuf[xcur])
    int32_t* y = nullptr;
    float* Xbuf[2] = {nullptr, nullptr};   // double-buffered inputs (mggcn_prefetch)
    int32_t* ybuf[2] = {nullptr, nullptr};
    float* T0 = nullptr;
    float* HWB = nullptr;
    float* BC[2] = {nullptr, nullptr};
    // stage groups (S > 1, see plan_groups): the remote blocks of one group are consumed by ONE
    // launch over a merged tile whose column t * max_rows_j + c addresses local column c of the
    // group's t-th block; the group's blocks land in consecutive BC slots packed at the SpMM's
    // width (slot k at BCg + k * max_rows_j * width), 2S slots (two groups in flight)
    float* BCg = nullptr;
    std::vector<HostTile> gF, gB;    // merged tiles per group (host)
    std::vector<HostItems> hgF, hgB;
    std::vector<SpmmTile> GF, GB;    // device
    std::vector<int32_t> order_cache;  // row order of the items (setup only)
    std::vector<float*> AHWB;
    float* spmm_partial = nullptr;
    double* ce_partial = nullptr;
    double* loss_local = nullptr;
    int64_t* ntrain_local = nullptr;
    float* WG_local = nullptr;
    float* gemm_partial = nullptr;
    cudaEvent_t ev_bc[2] = {nullptr, nullptr}, ev_free[2] = {nullptr, nullptr};
    // GEMM plans per layer: fwd (op 0), wgrad (op 2), igrad (op 1)
    std::vector<GemmPlan> g_fwd, g_wgrad, g_igrad;
    std::vector<int> has_fwd, has_wgrad, has_igrad;
};

}  // namespace

struct mggcn_model_s {
    int P = 1, nlocal = 1;          // P: row blocks of the partition (P' under MGGCN_F_REPL2)
    int c = 1;                      // replication factor (2 with MGGCN_F_REPL2)
    uint32_t flags = 0;
    int L = 0;
    std::vector<int64_t> d, ld;     // dims and padded leading dims (multiple of 4)
    std::vector<int> order;
    std::vector<int64_t> woff;      // per-layer offset into W/m/v/WG (floats)
    int64_t wtotal = 0;
    bool pattern = true;
    int64_t n_local = 0;            // rows owned by this model (sum over local ranks)
    int64_t max_rows_j = 0;
    int64_t bc_ld = 0, hw_ld = 0;
    // stage groups (choose_groups): remote indices [grp_b[g], grp_b[g+1]) are consumed by one
    // launch; empty = one launch per stage (the paper's schedule, BC1/BC2)
    std::vector<int> grp_b;
    bool grouped() const { return !grp_b.empty(); }
    std::vector<Rank> ranks;
    float *W = nullptr, *Mom = nullptr, *Vel = nullptr, *WG = nullptr;
    // tf32 hi/lo copies of W for the tcgen05 row GEMMs (refreshed after every update):
    // Wt_* = W^T [d_{l+1} x ld(d_l)] (B of Eq. 5), Ws_* = W [d_l x ld(d_{l+1})] (B of Eq. 11)
    std::vector<float*> Wt_hi, Wt_lo, Ws_hi, Ws_lo;
    double* loss_sum = nullptr;
    int64_t* ntrain = nullptr;
    cudaStream_t cs = nullptr, ms = nullptr;
    cudaEvent_t ev_begin = nullptr, ev_comm_end = nullptr, ev_tmp = nullptr, ev_wg = nullptr, ev_comm_done = nullptr;
    // without MGGCN_F_OVERLAP: recorded on the compute stream after every SpMM stage launch
    // (the local stage included); broadcast / pull k waits on it, so it starts only after
    // the previous stage finished (strict bcast -> stage -> bcast alternation)
    cudaEvent_t ev_stage = nullptr;
    ncclComm_t comm = nullptr;
    ncclComm_t comm_bc = nullptr, comm_pair = nullptr;   // 1.5D: replica group, row-block pair
    int state = ST_READY;
    int poisoned = 0;
    bool hung = false;              // a bounded host wait timed out: streams may never drain
    int64_t t = 0;
    bool need_wg_wait = false;
    // profiling
    std::vector<std::tuple<int, cudaEvent_t, cudaEvent_t>> prof_recs;
    std::vector<cudaEvent_t> prof_pool;
    // per-stage timeline (MGGCN_F_TIMELINE): {class, spmm index, stage, local rank, stream}, events
    struct TlRec { int32_t meta[5]; cudaEvent_t a, b; };
    std::vector<TlRec> tl_recs;
    int32_t tl_spmm = -1, tl_stage = -1, tl_rank = -1;   // context of the next ProfScope
    int32_t tl_nspmm = 0;                                  // SpMMs issued since the last forward
    double prof_ms[PC_N] = {0};
    int64_t prof_n[PC_N] = {0};
    // epoch work
    double w_spmm_bytes = 0, w_gather_bytes = 0, w_gemm_flops = 0, w_bcast_bytes = 0;
    double w_spmm_struct_bytes = 0, w_gemm_bytes = 0, w_ce_bytes = 0, w_gather_raw_bytes = 0, w_stages = 0;
    // X staging plan bookkeeping
    int layer_ids[64];
    bool t0_valid = false;          // MGGCN_F_CACHE_L0: T0 = Â'^T X computed
    // input prefetch (mggcn_prefetch): copy stream, staging chunk, buffer events
    // SM-free IPC exchange (MGGCN_F_IPC, NEXT-1): peers' workspaces, sequence flags
    uint32_t* flags_dev = nullptr;  // [0] spmm ready [1] spmm done [2] wg ready [3] wg done [4] sc ready [5] sc done
    float* WGp = nullptr;           // this rank's W_G partial (read by peers)
    char* ws_base = nullptr;        // this rank's workspace
    std::vector<char*> peer_ws;     // peers' workspaces mapped here (own = ws_base)
    std::vector<void*> ipc_opened;
    void* ipc_alloc = nullptr;
    size_t ipc_alloc_off = 0;
    bool ipc = false, ipc_connected = false;
    // dense blocks of the stage tiles (plan_dense): density threshold (MGGCN_DENSE_THR,
    // 0 = off) and bf16 pieces of the B operand (MGGCN_DENSE_PIECES, 2 or 3)
    double dense_thr = 0;
    double dense_min_frac = 0.5;    // MGGCN_DENSE_MINFRAC: blocks must hold this share of a tile's entries
    int64_t dense_min_rows = 0;     // MGGCN_DENSE_MIN_ROWS: ... in tiles of at least this many rows
    int64_t dense_min_entries = 0;  // MGGCN_DENSE_MIN_ENTRIES: ... and this many (coalesced) entries
    int dense_pieces = 3;
    // SOLO timing mode (MGGCN_F_NO_BCAST, P > 1, nlocal = 1, no NCCL id, no IPC): one rank of a
    // P-way run on its own, every collective skipped; per-rank compute time of a partition
    // too large for loopback (Papers-shaped at P = 8).  Results are invalid by construction.
    bool solo = false;
    // delay injection (mggcn_debug_comm_delay): spin kernels of pseudo-random length
    uint64_t delay_seed = 0, delay_ctr = 0;
    int32_t delay_max_us = 0;
    bool poison_bc = false;         // mggcn_debug_poison: NaN-fill every BC slot right before it is filled
    bool break_bc_wait = false;     // mggcn_debug_poison(m, 2): negative control, stages skip the broadcast wait
    size_t ws_bytes = 0;             // planned workspace bytes
    size_t sym_bytes = 0;            // symmetric region [0, sym_bytes) (IPC peers must agree)
    uint32_t spmm_seq = 0, wg_seq = 0, sc_seq = 0;
    cudaStream_t cp = nullptr;
    float* xstage = nullptr;
    int64_t xstage_floats = 0;
    cudaEvent_t ev_pref = nullptr, ev_xfree[2] = {nullptr, nullptr};
    int xcur = 0, pref_buf = -1;
    // captured epoch (mggcn_epoch_capture / mggcn_epoch_replay): forward -> backward -> step
    // as one CUDA graph; the Adam node's arguments are re-set per replay (step count t)
    bool capturing = false;
    cudaGraph_t eg = nullptr;
    cudaGraphExec_t ege = nullptr;
    cudaGraphNode_t eg_adam = nullptr;
    int64_t eg_kernels = 0;
    double eg_lr = 0, eg_b1 = 0, eg_b2 = 0, eg_eps = 0;
};

namespace {

#define CK(expr)                                                                                \
    do {                                                                                        \
        cudaError_t _e = (expr);                                                                \
        if (_e != cudaSuccess) {                                                                \
            set_error(std::string("CUDA error: ") + cudaGetErrorString(_e) + " at " #expr);     \
            return MGGCN_ECUDA;                                                                 \
        }                                                                                       \
    } while (0)

#define NK(expr)                                                                                \
    do {                                                                                        \
        ncclResult_t _r = (expr);                                                               \
        if (_r != ncclSuccess) {                                                                \
            set_error(std::string("NCCL error: ") + ncclGetErrorString(_r) + " at " #expr);     \
            return MGGCN_ENCCL;                                                                 \
        }                                                                                       \
    } while (0)

#define RC(expr)                         \
    do {                                 \
        int _rc = (expr);                \
        if (_rc != MGGCN_OK) return _rc; \
    } while (0)

// 1.5D: replica `rep` computes the stages of the column blocks j with j mod c == rep
inline bool in_set(const mggcn_model_s* m, int rep, int j) { return m->c == 1 || j % m->c == rep; }
// 1.5D: the replica of row block i that broadcasts it (i mod c) is its ROOT; only the root
// needs the block's GEMM products (HW, the input gradient) and contributes W_G, the loss and
// |T|; the other replica only adds its partial SpMM stages (every rank is a root in 1D)
inline bool is_root(const mggcn_model_s* m, const Rank& r) { return in_set(m, r.rep, r.rank); }

// The k-th remote block (k = 0 .. P-2) a rank consumes: ascending j != rank for the
// collective backends (broadcast order is global), rotated (rank + k + 1) mod P for the
// IPC pulls (every GPU serves one reader per step).
inline int remote_block(const mggcn_model_s* m, int rank, int k, bool ipc) {
    if (ipc) return (rank + k + 1) % m->P;
    return k < rank ? k : k + 1;
}
inline int n_groups(const mggcn_model_s* m) { return m->grouped() ? (int)m->grp_b.size() - 1 : 0; }
inline int group_of(const mggcn_model_s* m, int k) {
    int g = 0;
    while (k >= m->grp_b[g + 1]) ++g;
    return g;
}
inline bool last_of_group(const mggcn_model_s* m, int k) { return k == m->grp_b[group_of(m, k) + 1] - 1; }

// Stage groups.  One launch per stage (the paper's schedule) pays, per stage,
// a visit of every row with entries, an output read-modify-write, a launch
// and a hub fix-up; at P = 8 a Reddit-shaped rank's stages are 40-100 us, so
// these fixed costs are about a third of its SpMM time.  Grouped,
// the remote blocks get one BC slot each (P - 1 slots, no reuse inside a
// SpMM) and a group of them is consumed by ONE launch over a merged tile.
// The broadcasts then run back to back, so the SpMM ends at max(the compute
// chain, the last block's arrival + the LAST group's compute):
//  * compute-bound ranks (a block computes >= 1.5x longer than it takes to
//    arrive: e_row = coalesced entries per row per remote tile, compute / arrival
//    ~ e_row x 900 GB/s NVLink / 16 TB/s gathers >= 1.5, i.e. e_row >= 27; Reddit- and
//    Proteins-shaped at P = 8): two groups, ceil((P-1)/4) blocks (hidden behind the
//    local stage) and the rest;
//  * otherwise (Products-, Papers-shaped) the exchange bounds the SpMM, and the last
//    group's compute is exposed after the last arrival: groups (ceil((P-1)/4), middle, 1),
//    whose tail is one block, as in the per-stage schedule, with fewer launches.
// Off when the P - 1 slots exceed MGGCN_BC_BUDGET_MB (default 16 GiB: Papers-shaped
// 14 GB blocks keep BC1/BC2).  MGGCN_STAGE_GROUPS="a,b,.." (sizes summing to P - 1)
// or MGGCN_STAGE_GROUP=S (uniform; 1 = per stage) override.  1D only.
std::vector<int> choose_groups(const mggcn_model_s* m, double e_row) {
    std::vector<int> none;
    if (m->P <= 2 || m->c > 1) return none;
    if (const char* h = getenv("MGGCN_SPMM_HOTCLS"))
        if (atoi(h) != 0) return none;   // priority-class tiles keep per-stage launches
    const int R = m->P - 1;
    std::vector<int> sizes;
    if (const char* e = getenv("MGGCN_STAGE_GROUPS")) {
        int tot = 0;
        for (const char* c = e; *c;) {
            const int v = atoi(c);
            if (v <= 0) { sizes.clear(); break; }
            sizes.push_back(v);
            tot += v;
            while (*c && *c != ',') ++c;
            if (*c == ',') ++c;
        }
        if (tot != R) sizes.clear();
    }
    if (sizes.empty()) {
        int S = 0;
        if (const char* e = getenv("MGGCN_STAGE_GROUP")) S = atoi(e);
        if (S == 1) return none;
        if (S > 1) {
            for (int k = 0; k < R; k += S) sizes.push_back(std::min(S, R - k));
        } else {
            if (m->P < 4) return none;
            const int first = (R + 3) / 4;
            if (e_row * 900.0 / 16000.0 >= 1.5) sizes = {first, R - first};   // compute-bound
            else if (R - first >= 2) sizes = {first, R - first - 1, 1};      // exchange-bound
            else return none;
        }
    }
    double budget = 16384.0;
    if (const char* e = getenv("MGGCN_BC_BUDGET_MB")) budget = atof(e);
    const double slot_mb = (double)m->max_rows_j * (double)m->bc_ld * 4.0 / 1048576.0;
    if ((double)R * slot_mb > budget) return none;
    // merged column ids and the kernel's 32-bit float4 row offsets must not overflow
    if ((double)R * (double)m->max_rows_j * (double)(m->bc_ld / 4) >= 4294967296.0) return none;
    std::vector<int> b(1, 0);
    for (int v : sizes) b.push_back(b.back() + v);
    return b;
}

// ---------------------------------------------------------------- profiling
cudaEvent_t prof_event(mggcn_model_s* m) {
    if (!m->prof_pool.empty()) {
        cudaEvent_t e = m->prof_pool.back();
        m->prof_pool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}

// NVTX range names per op class (ranges for nsys / ncu --nvtx; no-ops without a tool)
const char* const kNvtxName[PC_N] = {"mggcn:spmm", "mggcn:gemm", "mggcn:loss", "mggcn:adam", "mggcn:bcast",
                                     "mggcn:allreduce", "mggcn:other", "mggcn:dense"};

struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};

struct ProfScope {
    NvtxRange nvtx;
    mggcn_model_s* m;
    int cls;
    cudaStream_t s;
    cudaEvent_t a = nullptr;     // MGGCN_F_PROFILE pair (consumed by mggcn_get_profile)
    cudaEvent_t ta = nullptr;    // MGGCN_F_TIMELINE pair (consumed by mggcn_get_timeline)
    int32_t meta[5];
    ProfScope(mggcn_model_s* m_, int c, cudaStream_t s_) : nvtx(kNvtxName[c]), m(m_), cls(c), s(s_) {
        if (m->capturing) return;   // a captured epoch is timed as a whole
        if (m->flags & MGGCN_F_PROFILE) {
            a = prof_event(m);
            cudaEventRecord(a, s);
        }
        if (m->flags & MGGCN_F_TIMELINE) {
            ta = prof_event(m);
            cudaEventRecord(ta, s);
            meta[0] = c;
            meta[1] = m->tl_spmm;
            meta[2] = m->tl_stage;
            meta[3] = m->tl_rank;
            meta[4] = s == m->cs ? 0 : 1;
        }
    }
    ~ProfScope() {
        if (a) {
            cudaEvent_t b = prof_event(m);
            cudaEventRecord(b, s);
            m->prof_recs.emplace_back(cls, a, b);
        }
        if (ta) {
            cudaEvent_t tb = prof_event(m);
            cudaEventRecord(tb, s);
            mggcn_model_s::TlRec t;
            for (int i = 0; i < 5; ++i) t.meta[i] = meta[i];
            t.a = ta;
            t.b = tb;
            m->tl_recs.push_back(t);
        }
    }
};

// --------------------------------------------------------------- planning
// 32-B (sector) aligned rows: narrow gathered rows (e.g. 41 -> 48 floats) stay sector aligned
int64_t ld_of(int64_t d) { return round_up(d, 8); }

int check_dims(int L, const int32_t* dims) {
    if (L < 1 || L > 64 || !dims) {
        set_error("model: L must be in [1, 64] and dims non-NULL");
        return MGGCN_EINVAL;
    }
    for (int l = 0; l <= L; ++l)
        if (dims[l] <= 0 || dims[l] > 65536) {
            set_error("model: every d_l must be in [1, 65536]");
            return MGGCN_EINVAL;
        }
    for (int l = 1; l < L; ++l)
        if (dims[l] < dims[l + 1] && true) {
            // SpMM-first at l > 0 (reading C22): needs a private T_l and a separate
            // mask buffer for the backward SpMM; no BASELINE config uses it.
            set_error("model: SpMM-first order (d_l < d_{l+1}) at layer l > 0 is not supported");
            return MGGCN_EUNSUPPORTED;
        }
    return MGGCN_OK;
}

// Lays out (or sizes, when bump.base == nullptr) every device buffer.
void plan_buffers(mggcn_model_s* m, Bump& b) {
    const int L = m->L;
    // ---- symmetric region: identical offsets on every rank of a multi-process run
    // (sizes use max_j n_j), so peers address each other's buffers by offset (IPC)
    m->flags_dev = b.take<uint32_t>(64);
    m->WGp = b.take<float>(m->wtotal);
    for (auto& r : m->ranks) {
        r.loss_local = b.take<double>(1);
        r.ntrain_local = b.take<int64_t>(1);
        for (int k = 0; k < 2; ++k) r.Xbuf[k] = b.take<float>(m->max_rows_j * m->ld[0]);
        r.HWB = b.take<float>(m->max_rows_j * std::max<int64_t>(m->hw_ld, 4));
        r.AHWB.assign(L, nullptr);
        for (int l = 0; l < L; ++l) r.AHWB[l] = b.take<float>(m->max_rows_j * m->ld[l + 1]);
    }
    m->sym_bytes = b.off;   // same on every rank (sizes use max_rows_j)
    // ---- private region
    m->W = b.take<float>(m->wtotal);
    m->Mom = b.take<float>(m->wtotal);
    m->Vel = b.take<float>(m->wtotal);
    m->WG = b.take<float>(m->wtotal);
    m->loss_sum = b.take<double>(1);
    m->ntrain = b.take<int64_t>(1);
    m->xstage_floats = (int64_t)16 << 20;   // 64 MB host-copy staging chunk for the copy stream
    m->xstage = b.take<float>(m->xstage_floats);
    m->Wt_hi.assign(L, nullptr); m->Wt_lo.assign(L, nullptr);
    m->Ws_hi.assign(L, nullptr); m->Ws_lo.assign(L, nullptr);
    for (int l = 0; l < L; ++l) {
        m->Wt_hi[l] = b.take<float>(m->d[l + 1] * m->ld[l]);
        m->Wt_lo[l] = b.take<float>(m->d[l + 1] * m->ld[l]);
        m->Ws_hi[l] = b.take<float>(m->d[l] * m->ld[l + 1]);
        m->Ws_lo[l] = b.take<float>(m->d[l] * m->ld[l + 1]);
    }
    for (auto& r : m->ranks) {
        const mggcn_part_s* pt = r.part;
        const int P = pt->P;
        r.F.assign(P, SpmmTile());
        r.B.assign(P, SpmmTile());
        auto place = [&](const HostTile& ht, const HostItems& hi, SpmmTile& t, bool hot_ok) {
            t.nrows = ht.nrows;
            t.ncols = ht.ncols;
            t.nnz = ht.rowptr.back();
            t.n_items = (int64_t)hi.items.size();
            t.n_items_nz = hi.n_nonempty;
            t.split = hi.split;
            t.n_splits = (int64_t)hi.splits.size();
            t.n_slots = hi.nslots;
            t.items = b.take<int4>(hi.items.size());
            t.splits = b.take<int4>(hi.splits.size());
            t.col = b.take<int32_t>(ht.col.size());
            t.hot_enc = hot_ok && want_hot_classes(ht);
            t.val = ht.val.empty() ? nullptr : b.take<float>(ht.val.size());
        };
        // dense blocks (device copies of a DenseHost); every tile shares the rank's B-image scratch
        size_t bimg_bytes = 0, part_floats = 0;
        auto place_dense = [&](const DenseHost& dh, SpmmTile& t) {
            t.dense = DenseTiles();
            if (!dh.active) return;
            DenseTiles& d = t.dense;
            d.n_groups = dh.n_groups;
            d.n_tiles = dh.n_tiles;
            d.n_chunks = dh.n_chunks;
            d.n_items = dh.n_items;
            d.n_splits = dh.n_splits;
            d.n_slots = dh.n_slots;
            d.n_bins = dh.n_bins;
            d.nnz = dh.nnz;
            d.pieces = m->dense_pieces;
            d.grp_rows = b.take<int32_t>(dh.grp_rows.size());
            d.row_flag = b.take<uint8_t>(dh.row_flag.size());
            d.work = b.take<int4>(dh.n_items);
            d.splits = b.take<int4>(dh.n_splits);
            d.bin_beg = b.take<int32_t>(dh.bin_beg.size());
            d.tile_chunk = b.take<int32_t>(dh.tile_chunk.size());
            d.chunk_cols = b.take<int32_t>(dh.chunk_cols.size());
            d.A = reinterpret_cast<const uint8_t*>(b.take<uint16_t>(dh.A.size()));
            bimg_bytes = std::max(bimg_bytes, dense_bimg_bytes(dh.n_chunks, m->dense_pieces));
            part_floats = std::max(part_floats, dense_partial_floats(dh.n_slots));
        };
        for (int j = 0; j < P; ++j) {
            // with stage groups only the local tile is launched per stage (the remote ones
            // live in the merged group tiles; mggcn_part_export_tile reads the host copies)
            const bool on_dev = !m->grouped() || j == r.rank;
            for (int dir = 0; dir < 2; ++dir) {
                if (dir == 1 && pt->shared_fb) {
                    r.B[j] = r.F[j];
                    continue;
                }
                SpmmTile& t = dir == 0 ? r.F[j] : r.B[j];
                if (on_dev) {
                    place(dir == 0 ? r.lF(j) : r.lB(j), dir == 0 ? r.hF[j] : r.hB[j], t, true);
                    const std::vector<DenseHost>& dv = dir == 0 ? r.dF : r.dB;
                    if (j < (int)dv.size()) place_dense(dv[j], t);
                }
            }
            if (pt->shared_fb) r.B[j] = r.F[j];
        }
        const int NG = n_groups(m);
        r.GF.assign(NG, SpmmTile());
        r.GB.assign(NG, SpmmTile());
        for (int g = 0; g < NG; ++g) {
            place(r.lgF(g), r.hgF[g], r.GF[g], false);
            if (g < (int)r.dgF.size()) place_dense(r.dgF[g], r.GF[g]);
            if (pt->shared_fb) r.GB[g] = r.GF[g];
            else {
                place(r.lgB(g), r.hgB[g], r.GB[g], false);
                if (g < (int)r.dgB.size()) place_dense(r.dgB[g], r.GB[g]);
            }
        }
        r.dense_bimg = bimg_bytes ? b.take<uint8_t>(bimg_bytes) : nullptr;
        r.dense_partial = part_floats ? b.take<float>(part_floats) : nullptr;
        for (auto* v : {&r.F, &r.B, &r.GF, &r.GB})
            for (auto& t : *v) {
                t.dense.bimg = r.dense_bimg;
                t.dense.partial = r.dense_partial;
            }
        r.inv_deg = b.take<float>(r.rows);
        for (int k = 0; k < 2; ++k) r.ybuf[k] = b.take<int32_t>(r.rows);
        r.Xs = r.Xbuf[0];
        r.y = r.ybuf[0];
        r.T0 = m->order[0] == S_ORDER ? b.take<float>(r.rows * m->ld[0]) : nullptr;
        if (P > 1 && !m->grouped()) {
            r.BC[0] = b.take<float>(m->max_rows_j * m->bc_ld);
            r.BC[1] = b.take<float>(m->max_rows_j * m->bc_ld);
        } else if (P > 1) {
            r.BCg = b.take<float>((P - 1) * m->max_rows_j * m->bc_ld);
        }
        int64_t slots = 0;
        for (int j = 0; j < P; ++j) {
            slots = std::max(slots, r.hF[j].nslots);
            if (!pt->shared_fb) slots = std::max(slots, r.hB[j].nslots);
        }
        for (int g = 0; g < NG; ++g) {
            slots = std::max(slots, r.hgF[g].nslots);
            if (!pt->shared_fb) slots = std::max(slots, r.hgB[g].nslots);
        }
        r.spmm_partial = b.take<float>(slots * std::min<int64_t>(m->bc_ld, 512));
        r.ce_partial = b.take<double>(kCeBlocks);
        r.WG_local = (m->nlocal > 1) ? b.take<float>(m->wtotal) : nullptr;
        // split-K partials for W_G (Eq. 10)
        size_t gp = 0;
        for (int l = 0; l < L; ++l)
            gp = std::max(gp, gemm_wgrad_partial_floats(m->d[l], m->d[l + 1], std::max<int64_t>(r.rows, 1)));
        r.gemm_partial = b.take<float>(gp);
    }
}

int upload_static(mggcn_model_s* m) {
    for (auto& r : m->ranks) {
        const mggcn_part_s* pt = r.part;
        auto upload = [&](const HostTile& ht, const HostItems& hi, SpmmTile& t) -> int {
                if (!hi.items.empty())
                    CK(cudaMemcpyAsync(const_cast<int4*>(t.items), hi.items.data(), sizeof(int4) * hi.items.size(),
                                       cudaMemcpyHostToDevice, m->cs));
                if (!hi.splits.empty())
                    CK(cudaMemcpyAsync(const_cast<int4*>(t.splits), hi.splits.data(),
                                       sizeof(int4) * hi.splits.size(), cudaMemcpyHostToDevice, m->cs));
                if (!ht.col.empty()) {
                    std::vector<int32_t> enc;
                    if (t.hot_enc) enc = encode_hot_classes(ht);
                    CK(cudaMemcpyAsync(const_cast<int32_t*>(t.col), t.hot_enc ? enc.data() : ht.col.data(),
                                       sizeof(int32_t) * ht.col.size(), cudaMemcpyHostToDevice, m->cs));
                    if (t.hot_enc) CK(cudaStreamSynchronize(m->cs));   // enc is a temporary
                }
                if (t.val && !ht.val.empty())
                    CK(cudaMemcpyAsync(const_cast<float*>(t.val), ht.val.data(), sizeof(float) * ht.val.size(),
                                       cudaMemcpyHostToDevice, m->cs));
                return MGGCN_OK;
        };
        auto upload_dense = [&](const DenseHost& dh, const SpmmTile& t) -> int {
            if (!dh.active) return MGGCN_OK;
            const DenseTiles& d = t.dense;
            auto cp = [&](const void* dst, const void* src, size_t bytes) -> int {
                if (bytes) CK(cudaMemcpyAsync(const_cast<void*>(dst), src, bytes, cudaMemcpyHostToDevice, m->cs));
                return MGGCN_OK;
            };
            RC(cp(d.grp_rows, dh.grp_rows.data(), 4 * dh.grp_rows.size()));
            RC(cp(d.row_flag, dh.row_flag.data(), dh.row_flag.size()));
            RC(cp(d.work, dh.work.data(), 4 * dh.work.size()));
            RC(cp(d.splits, dh.splits.data(), 4 * dh.splits.size()));
            RC(cp(d.bin_beg, dh.bin_beg.data(), 4 * dh.bin_beg.size()));
            RC(cp(d.tile_chunk, dh.tile_chunk.data(), 4 * dh.tile_chunk.size()));
            RC(cp(d.chunk_cols, dh.chunk_cols.data(), 4 * dh.chunk_cols.size()));
            RC(cp(d.A, dh.A.data(), 2 * dh.A.size()));
            return MGGCN_OK;
        };
        for (int j = 0; j < pt->P; ++j)
            for (int dir = 0; dir < 2; ++dir) {
                if (dir == 1 && pt->shared_fb) continue;
                if (m->grouped() && j != r.rank) continue;
                RC(upload(dir == 0 ? r.lF(j) : r.lB(j), dir == 0 ? r.hF[j] : r.hB[j], dir == 0 ? r.F[j] : r.B[j]));
                const std::vector<DenseHost>& dv = dir == 0 ? r.dF : r.dB;
                if (j < (int)dv.size()) RC(upload_dense(dv[j], dir == 0 ? r.F[j] : r.B[j]));
            }
        for (size_t g = 0; g < r.GF.size(); ++g) {
            RC(upload(r.lgF((int)g), r.hgF[g], r.GF[g]));
            if (g < r.dgF.size()) RC(upload_dense(r.dgF[g], r.GF[g]));
            if (!pt->shared_fb) {
                RC(upload(r.lgB((int)g), r.hgB[g], r.GB[g]));
                if (g < r.dgB.size()) RC(upload_dense(r.dgB[g], r.GB[g]));
            }
        }
        if (pt->shared_fb)
            for (int j = 0; j < pt->P; ++j) r.B[j] = r.F[j];
        if (pt->shared_fb)
            for (size_t g = 0; g < r.GF.size(); ++g) r.GB[g] = r.GF[g];
        CK(cudaMemcpyAsync(r.inv_deg, pt->inv_deg.data(), sizeof(float) * r.rows, cudaMemcpyHostToDevice, m->cs));
        // loopback W_G partials: the padding columns (ld > d) are summed with the rest (initcheck)
        if (r.WG_local) CK(cudaMemsetAsync(r.WG_local, 0, sizeof(float) * m->wtotal, m->cs));
        // zero every activation buffer once: padding columns stay 0 forever
        for (int k = 0; k < 2; ++k) CK(cudaMemsetAsync(r.Xbuf[k], 0, sizeof(float) * r.rows * m->ld[0], m->cs));
        for (int l = 0; l < m->L; ++l)
            CK(cudaMemsetAsync(r.AHWB[l], 0, sizeof(float) * r.rows * m->ld[l + 1], m->cs));
        CK(cudaMemsetAsync(r.HWB, 0, sizeof(float) * r.rows * std::max<int64_t>(m->hw_ld, 4), m->cs));
        if (r.T0) CK(cudaMemsetAsync(r.T0, 0, sizeof(float) * r.rows * m->ld[0], m->cs));
        for (int s = 0; s < 2; ++s)
            if (r.BC[s]) CK(cudaMemsetAsync(r.BC[s], 0, sizeof(float) * m->max_rows_j * m->bc_ld, m->cs));
        if (r.BCg) CK(cudaMemsetAsync(r.BCg, 0, sizeof(float) * (m->P - 1) * m->max_rows_j * m->bc_ld, m->cs));
    }
    CK(cudaMemsetAsync(m->W, 0, sizeof(float) * m->wtotal, m->cs));
    CK(cudaMemsetAsync(m->flags_dev, 0, sizeof(uint32_t) * 64, m->cs));
    CK(cudaMemsetAsync(m->WGp, 0, sizeof(float) * m->wtotal, m->cs));
    for (int l = 0; l < m->L; ++l) {
        CK(cudaMemsetAsync(m->Wt_hi[l], 0, sizeof(float) * m->d[l + 1] * m->ld[l], m->cs));
        CK(cudaMemsetAsync(m->Wt_lo[l], 0, sizeof(float) * m->d[l + 1] * m->ld[l], m->cs));
        CK(cudaMemsetAsync(m->Ws_hi[l], 0, sizeof(float) * m->d[l] * m->ld[l + 1], m->cs));
        CK(cudaMemsetAsync(m->Ws_lo[l], 0, sizeof(float) * m->d[l] * m->ld[l + 1], m->cs));
    }
    CK(cudaMemsetAsync(m->Mom, 0, sizeof(float) * m->wtotal, m->cs));
    CK(cudaMemsetAsync(m->Vel, 0, sizeof(float) * m->wtotal, m->cs));
    CK(cudaMemsetAsync(m->WG, 0, sizeof(float) * m->wtotal, m->cs));
    return MGGCN_OK;
}

// The input operand of layer l (H_l): staged X for l = 0, else H'_{l-1} in AHWB_{l-1}.
float* layer_input(mggcn_model_s* m, Rank& r, int l) { return l == 0 ? r.Xs : r.AHWB[l - 1]; }

// GEMM plans (tensor maps + tiling) of layer l for one rank; layer 0's depend
// on the current input buffer r.Xs and are rebuilt when it changes.
int plan_layer(mggcn_model_s* m, Rank& r, int l) {
    const int L = m->L;
    const int flags = (m->flags & MGGCN_F_TF32X1) ? GEMM_TF32X1 : 0;
    const bool relu_here = (l < L - 1) || (m->flags & MGGCN_F_RELU_LAST);
    // forward (Eq. 5): G-order HW = H W -> HWB ; S-order AHW = T W (+ReLU) -> AHWB_l
    if (m->order[l] == G_ORDER) {
        if (gemm_plan_rows(r.g_fwd[l], r.rows, m->d[l + 1], m->d[l], layer_input(m, r, l), m->ld[l], m->Wt_hi[l],
                           m->Wt_lo[l], m->ld[l], r.HWB, m->ld[l + 1], flags))
            return -1;
    } else {
        if (gemm_plan_rows(r.g_fwd[l], r.rows, m->d[l + 1], m->d[l], r.T0, m->ld[0], m->Wt_hi[l], m->Wt_lo[l],
                           m->ld[l], r.AHWB[l], m->ld[l + 1], flags | (relu_here ? GEMM_RELU : 0)))
            return -1;
    }
    r.has_fwd[l] = 1;
    // weight gradient (Eq. 10, reading C2): W_G = H^T HW_G (G) or T^T Z_G (S)
    {
        const float* Aop = m->order[l] == G_ORDER ? layer_input(m, r, l) : r.T0;
        const float* Bop = m->order[l] == G_ORDER ? r.HWB : r.AHWB[l];
        size_t pf = 0;
        if (gemm_plan_wgrad(r.g_wgrad[l], m->d[l], m->d[l + 1], r.rows, Aop, m->ld[l], Bop, m->ld[l + 1], flags, &pf))
            return -1;
        r.g_wgrad[l].partial = r.gemm_partial;
        r.has_wgrad[l] = 1;
    }
    // input gradient (Eq. 11) for l > 0: AHWB_{l-1} = (HW_G W^T) * [H'_{l-1} > 0] (* inv_deg)
    if (l > 0) {
        int f = flags | GEMM_MASK;
        if (m->order[l - 1] == G_ORDER && m->pattern) f |= GEMM_SCALE;
        if (gemm_plan_rows(r.g_igrad[l], r.rows, m->d[l], m->d[l + 1], r.HWB, m->ld[l + 1], m->Ws_hi[l],
                           m->Ws_lo[l], m->ld[l + 1], r.AHWB[l - 1], m->ld[l], f))
            return -1;
        r.g_igrad[l].rowscale = r.inv_deg;
        r.has_igrad[l] = 1;
    }
    return 0;
}

int plan_gemms(mggcn_model_s* m) {
    const int L = m->L;
    for (auto& r : m->ranks) {
        r.g_fwd.assign(L, GemmPlan());
        r.g_wgrad.assign(L, GemmPlan());
        r.g_igrad.assign(L, GemmPlan());
        r.has_fwd.assign(L, 0);
        r.has_wgrad.assign(L, 0);
        r.has_igrad.assign(L, 0);
        if (r.rows == 0) continue;
        for (int l = 0; l < L; ++l)
            if (plan_layer(m, r, l)) {
                set_error("model: GEMM plan / tensor-map encoding failed (needs an sm_100 device)");
                return MGGCN_ECUDA;
            }
    }
    return MGGCN_OK;
}

// Point every rank's layer-0 input at `Xrank(r)` and re-plan layer 0's GEMMs
// (tensor maps) if it changed.
template <typename F>
int set_layer0_input(mggcn_model_s* m, F Xrank) {
    for (auto& r : m->ranks) {
        float* x = Xrank(r);
        if (r.Xs == x) continue;
        r.Xs = x;
        if (r.rows && plan_layer(m, r, 0)) {
            set_error("model: GEMM re-plan failed");
            return MGGCN_ECUDA;
        }
    }
    return MGGCN_OK;
}

// Switch every rank to input buffer k (after a prefetch).
int use_input_buffer(mggcn_model_s* m, int k) {
    m->xcur = k;
    for (auto& r : m->ranks) r.y = r.ybuf[k];
    return set_layer0_input(m, [k](Rank& r) { return r.Xbuf[k]; });
}

// A device X with the padded row stride and 16-B alignment is used in place.
// IPC with a SpMM-first layer 0: the peers pull X from this rank's symmetric workspace at the
// offset of ITS current input buffer (peer_ptr), so X must live in Xbuf[xcur] (no zero-copy
// external pointer) and every rank must use the same buffer (no prefetch double-buffering).
bool ipc_x_exchanged(const mggcn_model_s* m) { return m->ipc && m->order[0] == S_ORDER && m->P > 1; }

bool device_zero_copy(mggcn_model_s* m, const float* X, int64_t ldx) {
    if (ipc_x_exchanged(m)) return false;
    if (ldx != m->ld[0] || (reinterpret_cast<uintptr_t>(X) & 15)) return false;
    cudaPointerAttributes pa;
    const bool dev = cudaPointerGetAttributes(&pa, X) == cudaSuccess && pa.type == cudaMemoryTypeDevice;
    cudaGetLastError();
    return dev;
}

int use_external_input(mggcn_model_s* m, const float* X) {
    for (auto& r : m->ranks) r.y = r.ybuf[m->xcur];
    return set_layer0_input(m, [&](Rank& r) { return const_cast<float*>(X) + r.row_off * m->ld[0]; });
}

// Input copy of (X, y) rows into buffer k on stream s (host or device source).
// A host X whose pitch differs from the padded ld goes through `stage` in
// contiguous chunks (1-D H2D, then a device 2-D copy): pitched H2D copies are slow.
int copy_inputs(mggcn_model_s* m, int k, const float* X, int64_t ldx, const int32_t* y, cudaStream_t s,
                float* stage, int64_t stage_floats) {
    cudaPointerAttributes pa;
    const bool host_x = cudaPointerGetAttributes(&pa, X) != cudaSuccess || pa.type == cudaMemoryTypeHost ||
                        pa.type == cudaMemoryTypeUnregistered;
    cudaGetLastError();   // clear a possible error from the attribute query
    for (auto& r : m->ranks) {
        if (r.rows == 0) continue;
        float* dst = r.Xbuf[k];
        if (host_x && ldx != m->ld[0]) {
            const int64_t chunk = std::max<int64_t>(1, stage_floats / ldx);
            for (int64_t r0 = 0; r0 < r.rows; r0 += chunk) {
                const int64_t nr = std::min(chunk, r.rows - r0);
                CK(cudaMemcpyAsync(stage, X + (r.row_off + r0) * ldx, sizeof(float) * nr * ldx,
                                   cudaMemcpyHostToDevice, s));
                CK(cudaMemcpy2DAsync(dst + r0 * m->ld[0], m->ld[0] * 4, stage, ldx * 4, m->d[0] * 4, nr,
                                     cudaMemcpyDeviceToDevice, s));
            }
        } else if (ldx == m->ld[0]) {
            // already in the padded layout (host or device): one contiguous copy; the padding
            // columns are copied too and never read as data (GEMM tensor maps stop at d_0)
            CK(cudaMemcpyAsync(dst, X + r.row_off * ldx, sizeof(float) * r.rows * ldx, cudaMemcpyDefault, s));
        } else {
            CK(cudaMemcpy2DAsync(dst, m->ld[0] * 4, X + r.row_off * ldx, ldx * 4, m->d[0] * 4, r.rows,
                                 cudaMemcpyDefault, s));
        }
        CK(cudaMemcpyAsync(r.ybuf[k], y + r.row_off, sizeof(int32_t) * r.rows, cudaMemcpyDefault, s));
    }
    return MGGCN_OK;
}

// tf32 hi / lo weight copies for the row GEMMs (after set_weights and Adam).
int refresh_weight_splits(mggcn_model_s* m) {
    const int x1 = (m->flags & MGGCN_F_TF32X1) ? 1 : 0;
    for (int l = 0; l < m->L; ++l)
        CK(launch_split_weights(m->W + m->woff[l], m->d[l], m->d[l + 1], m->ld[l + 1], m->Wt_hi[l], m->Wt_lo[l],
                                m->ld[l], m->Ws_hi[l], m->Ws_lo[l], x1, m->cs));
    return MGGCN_OK;
}

// --------------------------------------------------------------------- IPC
// Address of `mine` (a buffer in this rank's symmetric region) inside peer q.
template <typename T>
T* peer_ptr(mggcn_model_s* m, int q, T* mine) {
    return reinterpret_cast<T*>(m->peer_ws[q] + (reinterpret_cast<char*>(mine) - m->ws_base));
}

int ipc_signal(mggcn_model_s* m, cudaStream_t s, int flag, uint32_t seq) {
    CK(stream_write_u32(s, m->flags_dev + flag, seq));
    return MGGCN_OK;
}

// stream s waits until every peer's flag >= seq
int ipc_wait_peers(mggcn_model_s* m, cudaStream_t s, int flag, uint32_t seq) {
    const int me = m->ranks[0].rank;
    for (int q = 0; q < m->P; ++q)
        if (q != me) CK(stream_wait_u32(s, peer_ptr(m, q, m->flags_dev) + flag, seq));
    return MGGCN_OK;
}

// --------------------------------------------------------- staged SpMM
// C_r (+)= sum_j T_rj · S_j over stages; S_j = src(j) rows of rank j.
// Local stage first, then ascending j (reading C13); broadcast q goes into
// BC[k % 2] for the k-th remote stage; broadcast k waits for the SpMM of
// remote stage k-2; SpMM k waits for broadcast k.
struct SpmmJob {
    int dir;                 // 0: F tiles (Â'^T), 1: B tiles (Â')
    int64_t width;           // = ld of src/out (multiple of 4)
    bool use_rowscale;       // inv_deg of the output row on the last stage
    bool relu;
    float* (*src)(mggcn_model_s*, Rank&, const void*);
    float* (*dst)(mggcn_model_s*, Rank&, const void*);
    const void* ctx;
};

// delay injection: a spin of 0..delay_max_us on stream s (test hook, P:929-941 rule check)
int inject_delay(mggcn_model_s* m, cudaStream_t s) {
    if (m->delay_max_us <= 0) return MGGCN_OK;
    if (m->break_bc_wait && s == m->cs) return MGGCN_OK;   // negative control: only the exchange is late
    uint64_t z = m->delay_seed + 0x9E3779B97F4A7C15ull * (++m->delay_ctr);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    z ^= z >> 31;
    CK(launch_spin((z % ((uint64_t)m->delay_max_us + 1)) * 1000ull, s));
    return MGGCN_OK;
}

// poison-buffer injection (mggcn_debug_poison): the comm stream NaN-fills a BC slot right
// before the broadcast / copy / pull into it, so a stage that read a slot outside the
// P:939-941 event rule would turn its rows into NaN instead of silently reading stale data
int poison_slot(mggcn_model_s* m, void* p, size_t bytes) {
    if (m->poison_bc && bytes) CK(cudaMemsetAsync(p, 0xFF, bytes, m->ms));
    return MGGCN_OK;
}

// compute-stream wait for a broadcast / pull (skipped only by the negative-control hook)
int wait_bc(mggcn_model_s* m, cudaEvent_t e) {
    if (!m->break_bc_wait) CK(cudaStreamWaitEvent(m->cs, e, 0));
    return MGGCN_OK;
}

// One SpMM stage launch: the dense blocks under their own PC_DENSE scope (nested in the
// caller's PC_SPMM scope), then the gather of the residual entries.
cudaError_t spmm_call(mggcn_model_s* m, const SpmmTile& t, const float* B, int width, float* out, float* partial,
                      const float* rowscale, int flags) {
    if (t.dense.n_items > 0) {
        ProfScope pd(m, PC_DENSE, m->cs);
        cudaError_t e = launch_spmm_dense(t, B, width, out, width, width, flags, m->cs);
        if (e != cudaSuccess) return e;
    }
    return launch_spmm_gather(t, B, width, out, width, partial, rowscale, width, flags, m->cs);
}

int launch_stage(mggcn_model_s* m, Rank& r, const SpmmJob& job, int j, const float* B, int flags, int tl_k) {
    RC(inject_delay(m, m->cs));
    const SpmmTile& t = job.dir == 0 ? r.F[j] : r.B[j];
    float* out = job.dst(m, r, job.ctx);
    m->tl_stage = tl_k;
    m->tl_rank = (int32_t)(&r - &m->ranks[0]);
    ProfScope ps(m, PC_SPMM, m->cs);
    // NCCL collectives run as kernels on the comm stream: let them in while the SpMM runs
    if ((m->comm || m->solo) && m->P > 1 && (m->flags & MGGCN_F_OVERLAP)) flags |= SPMM_YIELD;
    CK(spmm_call(m, t, B, (int)job.width, out, r.spmm_partial, job.use_rowscale ? r.inv_deg : nullptr,
                 flags | (job.relu ? SPMM_RELU : 0)));
    return MGGCN_OK;
}

// Without MGGCN_F_OVERLAP the exchange of block k may start only after the
// previous SpMM stage (the local stage for k = 0) finished: mark_stage() after
// every stage launch, serial_wait() before every broadcast / pull.
int mark_stage(mggcn_model_s* m) {
    if (!(m->flags & MGGCN_F_OVERLAP)) CK(cudaEventRecord(m->ev_stage, m->cs));
    return MGGCN_OK;
}
int serial_wait(mggcn_model_s* m) {
    if (!(m->flags & MGGCN_F_OVERLAP)) CK(cudaStreamWaitEvent(m->ms, m->ev_stage, 0));
    return MGGCN_OK;
}
// timeline context of a broadcast / pull ProfScope
void tl_comm(mggcn_model_s* m, int k, int rank_idx) {
    m->tl_stage = k;
    m->tl_rank = rank_idx;
}

int remote_index(int q, int self) { return q < self ? q : q - 1; }

// Stage groups (choose_groups): remote index k of a rank lands in its own slot k,
// packed at the SpMM's width, so a group's blocks are one contiguous operand for
// its merged tile.
float* group_slot(mggcn_model_s* m, Rank& r, int k, int64_t width) {
    return r.BCg + (size_t)k * (size_t)m->max_rows_j * (size_t)width;
}

int launch_group(mggcn_model_s* m, Rank& r, const SpmmJob& job, int g, int flags, int tl_k) {
    RC(inject_delay(m, m->cs));
    const SpmmTile& t = job.dir == 0 ? r.GF[g] : r.GB[g];
    float* out = job.dst(m, r, job.ctx);
    m->tl_stage = tl_k;
    m->tl_rank = (int32_t)(&r - &m->ranks[0]);
    ProfScope ps(m, PC_SPMM, m->cs);
    if ((m->comm || m->solo) && m->P > 1 && (m->flags & MGGCN_F_OVERLAP)) flags |= SPMM_YIELD;
    const float* B = group_slot(m, r, m->grp_b[g], job.width);
    CK(spmm_call(m, t, B, (int)job.width, out, r.spmm_partial, job.use_rowscale ? r.inv_deg : nullptr,
                 flags | (job.relu ? SPMM_RELU : 0)));
    return MGGCN_OK;
}

// NEXT-1 (SM-free exchange): every receiver PULLS the peers' blocks with copy
// engines in rotated order (stage s reads block (i + s) mod P, so each GPU
// serves one reader per step); sequence flags order producer -> pull -> reuse.
int staged_spmm_ipc(mggcn_model_s* m, const SpmmJob& job) {
    const int P = m->P;
    Rank& r = m->ranks[0];
    const int me = r.rank;
    const uint32_t seq = ++m->spmm_seq;
    const bool nob = (m->flags & MGGCN_F_NO_BCAST) != 0;
    float* mysrc = job.src(m, r, job.ctx);
    CK(cudaEventRecord(m->ev_begin, m->cs));            // my source produced; BC slots free
    RC(ipc_signal(m, m->cs, 0, seq));                   // peers may pull my block
    CK(cudaStreamWaitEvent(m->ms, m->ev_begin, 0));
    if (r.rows > 0) RC(launch_stage(m, r, job, me, mysrc, 0, -1));
    RC(mark_stage(m));
    if (m->grouped()) {   // stage groups: pulls into dedicated slots, one launch per group
        const int NG = n_groups(m);
        for (int k = 0; k < P - 1; ++k) {
            const int q = (me + k + 1) % P, g = group_of(m, k);
            const bool last = last_of_group(m, k);
            {
                RC(serial_wait(m));
                tl_comm(m, q, 0);
                ProfScope ps(m, PC_BCAST, m->ms);
                RC(inject_delay(m, m->ms));
                CK(stream_wait_u32(m->ms, peer_ptr(m, q, m->flags_dev) + 0, seq));   // block q is ready
                const size_t bytes = (size_t)(r.part->p[q + 1] - r.part->p[q]) * (size_t)job.width * sizeof(float);
                if (!nob && bytes) RC(poison_slot(m, group_slot(m, r, k, job.width), bytes));
                if (!nob && bytes)
                    CK(cudaMemcpyAsync(group_slot(m, r, k, job.width), peer_ptr(m, q, mysrc), bytes, cudaMemcpyDefault,
                                       m->ms));
                if (last) CK(cudaEventRecord(r.ev_bc[g & 1], m->ms));
            }
            if (last) {
                RC(wait_bc(m, r.ev_bc[g & 1]));
                if (r.rows > 0) RC(launch_group(m, r, job, g, SPMM_ACCUM | (g == NG - 1 ? SPMM_LAST : 0), q));
                RC(mark_stage(m));
            }
        }
    } else
    for (int st = 1; st < P; ++st) {
        const int q = (me + st) % P, k = st - 1, slot = k & 1;
        {
            RC(serial_wait(m));
            tl_comm(m, q, 0);
            ProfScope ps(m, PC_BCAST, m->ms);
            RC(inject_delay(m, m->ms));
            if (k >= 2) CK(cudaStreamWaitEvent(m->ms, r.ev_free[slot], 0));
            CK(stream_wait_u32(m->ms, peer_ptr(m, q, m->flags_dev) + 0, seq));   // block q is ready
            const size_t bytes = (size_t)(r.part->p[q + 1] - r.part->p[q]) * (size_t)job.width * sizeof(float);
            if (!nob && bytes) RC(poison_slot(m, r.BC[slot], bytes));
            if (!nob && bytes) CK(cudaMemcpyAsync(r.BC[slot], peer_ptr(m, q, mysrc), bytes, cudaMemcpyDefault, m->ms));
            CK(cudaEventRecord(r.ev_bc[slot], m->ms));
        }
        RC(wait_bc(m, r.ev_bc[slot]));
        if (r.rows > 0) RC(launch_stage(m, r, job, q, r.BC[slot], SPMM_ACCUM | (st == P - 1 ? SPMM_LAST : 0), q));
        CK(cudaEventRecord(r.ev_free[slot], m->cs));
        RC(mark_stage(m));
    }
    RC(ipc_signal(m, m->ms, 1, seq));                   // I have read every peer's block
    CK(cudaEventRecord(m->ev_comm_end, m->ms));
    CK(cudaStreamWaitEvent(m->cs, m->ev_comm_end, 0));
    RC(ipc_wait_peers(m, m->cs, 1, seq));               // ... and the peers have read mine
    return MGGCN_OK;
}

// 1.5D (c = 2): rank (i, r) runs the stages of
// the column blocks j in J_r = {j : j mod c = r} (its own block first when
// i is in J_r, then ascending j); block j is broadcast by rank (j, r) inside
// replica group r only, into BC[k % 2] for the k-th remote stage with the
// same slot rule as the 1D schedule.  No stage applies the last-stage
// epilogue: the two replicas' partial sums are added (NCCL all-reduce over
// the row-block pair, or one loopback kernel per pair writing both copies)
// and then scaled by 1/deg (Eq. 2) and passed through ReLU (Eq. 7).
int remote_index_15d(const mggcn_model_s* m, int q, const Rank& r) {
    int k = 0;
    for (int j = 0; j < q; ++j)
        if (j != r.rank && in_set(m, r.rep, j)) ++k;
    return k;
}

int staged_spmm_15d(mggcn_model_s* m, const SpmmJob& job) {
    const int P = m->P, c = m->c;
    const bool nob = (m->flags & MGGCN_F_NO_BCAST) != 0;
    CK(cudaEventRecord(m->ev_begin, m->cs));
    CK(cudaStreamWaitEvent(m->ms, m->ev_begin, 0));
    std::vector<char> started(m->ranks.size(), 0);
    for (size_t k = 0; k < m->ranks.size(); ++k) {      // own block first
        Rank& r = m->ranks[k];
        if (!in_set(m, r.rep, r.rank)) continue;
        if (r.rows > 0) RC(launch_stage(m, r, job, r.rank, job.src(m, r, job.ctx), 0, -1));
        started[k] = 1;
    }
    RC(mark_stage(m));
    for (int q = 0; q < P; ++q) {
        const int rq = q % c;                            // the replica group that needs block q
        {
            RC(serial_wait(m));
            tl_comm(m, q, -1);
            ProfScope ps(m, PC_BCAST, m->ms);
            RC(inject_delay(m, m->ms));
            if (m->comm || m->solo) {   // solo: nob is set, only the slot events remain
                Rank& r = m->ranks[0];
                if (r.rep == rq) {
                    const size_t count = (size_t)(r.part->p[q + 1] - r.part->p[q]) * (size_t)job.width;
                    if (q == r.rank) {
                        float* s = job.src(m, r, job.ctx);
                        if (!nob && count) NK(ncclBroadcast(s, s, count, ncclFloat32, q, m->comm_bc, m->ms));
                    } else {
                        const int k = remote_index_15d(m, q, r), slot = k & 1;
                        if (k >= 2) CK(cudaStreamWaitEvent(m->ms, r.ev_free[slot], 0));
                        if (!nob && count) RC(poison_slot(m, r.BC[slot], count * sizeof(float)));
                        if (!nob && count)
                            NK(ncclBroadcast(r.BC[slot], r.BC[slot], count, ncclFloat32, q, m->comm_bc, m->ms));
                        CK(cudaEventRecord(r.ev_bc[slot], m->ms));
                    }
                }
            } else {
                Rank& root = m->ranks[rq * P + q];
                const size_t bytes = (size_t)root.rows * (size_t)job.width * sizeof(float);
                for (auto& r : m->ranks) {
                    if (r.rep != rq || r.rank == q) continue;
                    const int k = remote_index_15d(m, q, r), slot = k & 1;
                    if (k >= 2) CK(cudaStreamWaitEvent(m->ms, r.ev_free[slot], 0));
                    if (!nob && bytes) RC(poison_slot(m, r.BC[slot], bytes));
                    if (!nob && bytes)
                        CK(cudaMemcpyAsync(r.BC[slot], job.src(m, root, job.ctx), bytes, cudaMemcpyDeviceToDevice,
                                           m->ms));
                    CK(cudaEventRecord(r.ev_bc[slot], m->ms));
                }
            }
        }
        for (size_t i = 0; i < m->ranks.size(); ++i) {
            Rank& r = m->ranks[i];
            if (r.rep != rq || r.rank == q) continue;
            const int k = remote_index_15d(m, q, r), slot = k & 1;
            RC(wait_bc(m, r.ev_bc[slot]));
            if (r.rows > 0) RC(launch_stage(m, r, job, q, r.BC[slot], started[i] ? SPMM_ACCUM : 0, q));
            started[i] = 1;
            CK(cudaEventRecord(r.ev_free[slot], m->cs));
        }
        RC(mark_stage(m));
    }
    CK(cudaEventRecord(m->ev_comm_end, m->ms));
    CK(cudaStreamWaitEvent(m->cs, m->ev_comm_end, 0));
    // ---- pair reduction of the replicas' partial sums, then the last-stage epilogue
    const int relu = job.relu ? 1 : 0;
    if (m->comm) {
        Rank& r = m->ranks[0];
        float* out = job.dst(m, r, job.ctx);
        CK(cudaEventRecord(m->ev_tmp, m->cs));
        CK(cudaStreamWaitEvent(m->ms, m->ev_tmp, 0));
        {
            ProfScope ps(m, PC_ALLRED, m->ms);
            if (r.rows) NK(ncclAllReduce(out, out, (size_t)r.rows * (size_t)job.width, ncclFloat32, ncclSum,
                                         m->comm_pair, m->ms));
        }
        CK(cudaEventRecord(m->ev_tmp, m->ms));
        CK(cudaStreamWaitEvent(m->cs, m->ev_tmp, 0));
        ProfScope ps(m, PC_SPMM, m->cs);
        CK(launch_rows_epilogue(out, r.rows, (int)job.width, job.width, job.use_rowscale ? r.inv_deg : nullptr, relu,
                                m->cs));
    } else {
        ProfScope ps(m, PC_SPMM, m->cs);
        for (int i = 0; i < P; ++i) {
            Rank& a = m->ranks[i];
            Rank& b = m->ranks[P + i];
            CK(launch_pair_sum_epilogue(job.dst(m, a, job.ctx), job.dst(m, b, job.ctx), a.rows, (int)job.width,
                                        job.width, job.use_rowscale ? a.inv_deg : nullptr, relu, m->cs));
        }
    }
    return MGGCN_OK;
}

// 1D schedule with stage groups: the broadcasts keep their global order
// (q = 0..P-1, every rank joins every collective); a rank launches group g
// once the last block of g has arrived; group g + 2 reuses group g's slots.
int staged_spmm_grouped(mggcn_model_s* m, const SpmmJob& job) {
    const int P = m->P, NG = n_groups(m);
    const bool nob = (m->flags & MGGCN_F_NO_BCAST) != 0;
    for (auto& r : m->ranks)
        if (r.rows > 0) RC(launch_stage(m, r, job, r.rank, job.src(m, r, job.ctx), 0, -1));
    RC(mark_stage(m));
    for (int q = 0; q < P; ++q) {
        {
            RC(serial_wait(m));
            tl_comm(m, q, -1);
            ProfScope ps(m, PC_BCAST, m->ms);
            RC(inject_delay(m, m->ms));
            if (m->comm || m->solo) {   // solo: nob is set, only the slot events remain
                Rank& r = m->ranks[0];
                const size_t count = (size_t)(r.part->p[q + 1] - r.part->p[q]) * (size_t)job.width;
                if (q == r.rank) {
                    float* src = job.src(m, r, job.ctx);
                    if (!nob && count) NK(ncclBroadcast(src, src, count, ncclFloat32, q, m->comm, m->ms));
                } else {
                    const int k = remote_index(q, r.rank);
                    float* dst = group_slot(m, r, k, job.width);
                    if (!nob && count) RC(poison_slot(m, dst, count * sizeof(float)));
                    if (!nob && count) NK(ncclBroadcast(dst, dst, count, ncclFloat32, q, m->comm, m->ms));
                    if (last_of_group(m, k)) CK(cudaEventRecord(r.ev_bc[group_of(m, k) & 1], m->ms));
                }
            } else {
                Rank& root = m->ranks[q];
                const size_t bytes = (size_t)root.rows * (size_t)job.width * sizeof(float);
                for (auto& r : m->ranks) {
                    if (r.rank == q) continue;
                    const int k = remote_index(q, r.rank);
                    if (!nob && bytes) RC(poison_slot(m, group_slot(m, r, k, job.width), bytes));
                    if (!nob && bytes)
                        CK(cudaMemcpyAsync(group_slot(m, r, k, job.width), job.src(m, root, job.ctx), bytes,
                                           cudaMemcpyDeviceToDevice, m->ms));
                    if (last_of_group(m, k)) CK(cudaEventRecord(r.ev_bc[group_of(m, k) & 1], m->ms));
                }
            }
        }
        for (auto& r : m->ranks) {
            if (r.rank == q) continue;
            const int k = remote_index(q, r.rank);
            if (!last_of_group(m, k)) continue;
            const int g = group_of(m, k);
            RC(wait_bc(m, r.ev_bc[g & 1]));
            if (r.rows > 0) RC(launch_group(m, r, job, g, SPMM_ACCUM | (g == NG - 1 ? SPMM_LAST : 0), q));
        }
        RC(mark_stage(m));
    }
    CK(cudaEventRecord(m->ev_comm_end, m->ms));
    CK(cudaStreamWaitEvent(m->cs, m->ev_comm_end, 0));
    return MGGCN_OK;
}

int staged_spmm_impl(mggcn_model_s* m, const SpmmJob& job) {
    if (m->c > 1) return staged_spmm_15d(m, job);
    const int P = m->P;
    const bool nob = (m->flags & MGGCN_F_NO_BCAST) != 0;
    if (P > 1) {
        CK(cudaEventRecord(m->ev_begin, m->cs));
        CK(cudaStreamWaitEvent(m->ms, m->ev_begin, 0));
    }
    if (m->ipc) return staged_spmm_ipc(m, job);
    if (m->grouped()) return staged_spmm_grouped(m, job);
    // local stage
    for (auto& r : m->ranks) {
        if (r.rows == 0) continue;
        const int last = (P == 1) ? SPMM_LAST : 0;
        RC(launch_stage(m, r, job, r.rank, job.src(m, r, job.ctx), last, -1));
    }
    if (P == 1) return MGGCN_OK;
    RC(mark_stage(m));
    for (int q = 0; q < P; ++q) {
        // ---- broadcast of block q (comm stream)
        {
            RC(serial_wait(m));
            tl_comm(m, q, -1);
            ProfScope ps(m, PC_BCAST, m->ms);
            RC(inject_delay(m, m->ms));
            if (m->comm || m->solo) {   // solo: nob is set, only the slot events remain
                Rank& r = m->ranks[0];
                const size_t count = (size_t)(r.part->p[q + 1] - r.part->p[q]) * (size_t)job.width;
                if (q == r.rank) {
                    float* s = job.src(m, r, job.ctx);
                    if (!nob && count) NK(ncclBroadcast(s, s, count, ncclFloat32, q, m->comm, m->ms));
                } else {
                    const int k = remote_index(q, r.rank), slot = k & 1;
                    if (k >= 2) CK(cudaStreamWaitEvent(m->ms, r.ev_free[slot], 0));
                    if (!nob && count) RC(poison_slot(m, r.BC[slot], count * sizeof(float)));
                    if (!nob && count) NK(ncclBroadcast(r.BC[slot], r.BC[slot], count, ncclFloat32, q, m->comm, m->ms));
                    CK(cudaEventRecord(r.ev_bc[slot], m->ms));
                }
            } else {
                Rank& root = m->ranks[q];
                const size_t bytes = (size_t)root.rows * (size_t)job.width * sizeof(float);
                for (auto& r : m->ranks) {
                    if (r.rank == q) continue;
                    const int k = remote_index(q, r.rank), slot = k & 1;
                    if (k >= 2) CK(cudaStreamWaitEvent(m->ms, r.ev_free[slot], 0));
                    if (!nob && bytes) RC(poison_slot(m, r.BC[slot], bytes));
                    if (!nob && bytes)
                        CK(cudaMemcpyAsync(r.BC[slot], job.src(m, root, job.ctx), bytes, cudaMemcpyDeviceToDevice,
                                           m->ms));
                    CK(cudaEventRecord(r.ev_bc[slot], m->ms));
                }
            }
        }
        // ---- SpMM stage q on every local receiver (compute stream)
        for (auto& r : m->ranks) {
            if (r.rank == q) continue;
            const int k = remote_index(q, r.rank), slot = k & 1;
            RC(wait_bc(m, r.ev_bc[slot]));
            const int last_q = (r.rank == P - 1) ? P - 2 : P - 1;
            const int flags = SPMM_ACCUM | (q == last_q ? SPMM_LAST : 0);
            if (r.rows > 0) RC(launch_stage(m, r, job, q, r.BC[slot], flags, q));
            CK(cudaEventRecord(r.ev_free[slot], m->cs));
        }
        RC(mark_stage(m));
    }
    CK(cudaEventRecord(m->ev_comm_end, m->ms));
    CK(cudaStreamWaitEvent(m->cs, m->ev_comm_end, 0));
    return MGGCN_OK;
}

int staged_spmm(mggcn_model_s* m, const SpmmJob& job) {
    m->tl_spmm = m->tl_nspmm++;
    const int rc = staged_spmm_impl(m, job);
    m->tl_spmm = m->tl_stage = m->tl_rank = -1;
    return rc;
}

float* src_HWB(mggcn_model_s*, Rank& r, const void*) { return r.HWB; }
float* src_X(mggcn_model_s*, Rank& r, const void*) { return r.Xs; }
float* src_T0(mggcn_model_s*, Rank& r, const void*) { return r.T0; }
float* src_AHWB(mggcn_model_s*, Rank& r, const void* ctx) { return r.AHWB[*static_cast<const int*>(ctx)]; }

// Tiny reductions across ranks (loss, |T|) for nlocal == 1: NCCL all-reduce
// on the comm stream fenced by events, or a copy when P == 1.
int reduce_scalars(mggcn_model_s* m, bool ntrain) {
    Rank& r = m->ranks[0];
    if (m->ipc) {
        // every rank sums all P partials in rank order (identical results on all ranks)
        const uint32_t seq = ++m->sc_seq;
        RC(ipc_signal(m, m->cs, 4, seq));
        RC(ipc_wait_peers(m, m->cs, 4, seq));
        std::vector<const double*> pd(m->P);
        std::vector<const int64_t*> pi(m->P);
        for (int q = 0; q < m->P; ++q) {
            pd[q] = peer_ptr(m, q, r.loss_local);
            pi[q] = peer_ptr(m, q, r.ntrain_local);
        }
        if (ntrain) CK(launch_sum_ranks_scalar(nullptr, pi.data(), m->P, nullptr, m->ntrain, m->cs));
        else CK(launch_sum_ranks_scalar(pd.data(), nullptr, m->P, m->loss_sum, nullptr, m->cs));
        RC(ipc_signal(m, m->cs, 5, seq));
    } else if (m->comm) {
        CK(cudaEventRecord(m->ev_tmp, m->cs));
        CK(cudaStreamWaitEvent(m->ms, m->ev_tmp, 0));
        if (ntrain) NK(ncclAllReduce(r.ntrain_local, m->ntrain, 1, ncclInt64, ncclSum, m->comm, m->ms));
        else NK(ncclAllReduce(r.loss_local, m->loss_sum, 1, ncclFloat64, ncclSum, m->comm, m->ms));
        CK(cudaEventRecord(m->ev_tmp, m->ms));
        CK(cudaStreamWaitEvent(m->cs, m->ev_tmp, 0));
    } else if (ntrain) {
        CK(cudaMemcpyAsync(m->ntrain, r.ntrain_local, 8, cudaMemcpyDeviceToDevice, m->cs));
    } else {
        CK(cudaMemcpyAsync(m->loss_sum, r.loss_local, 8, cudaMemcpyDeviceToDevice, m->cs));
    }
    return MGGCN_OK;
}

}  // namespace

// Loopback scalar reduction with an explicit ordered kernel over gathered values.
static int reduce_scalars_loopback(mggcn_model_s* m, bool ntrain) {
    // gather into a contiguous scratch (the first rank's ce_partial has room: kCeBlocks doubles)
    const int R = (int)m->ranks.size();
    double* scratch = m->ranks[0].ce_partial;   // free between loss passes (consumed already)
    for (int i = 0; i < R; ++i) {
        if (ntrain)
            CK(cudaMemcpyAsync(reinterpret_cast<int64_t*>(scratch) + i, m->ranks[i].ntrain_local, 8,
                               cudaMemcpyDeviceToDevice, m->cs));
        else
            CK(cudaMemcpyAsync(scratch + i, m->ranks[i].loss_local, 8, cudaMemcpyDeviceToDevice, m->cs));
    }
    if (ntrain) CK(launch_sum_i64(reinterpret_cast<int64_t*>(scratch), R, m->ntrain, m->cs));
    else CK(launch_sum_f64(scratch, R, m->loss_sum, m->cs));
    return MGGCN_OK;
}

static int reduce_all(mggcn_model_s* m, bool ntrain) {
    if (m->nlocal > 1) return reduce_scalars_loopback(m, ntrain);
    return reduce_scalars(m, ntrain);
}

static int poison(mggcn_model_s* m, int rc) {
    if (rc == MGGCN_ECUDA || rc == MGGCN_ENCCL) m->poisoned = rc;
    return rc;
}

// ------------------------------------------------- bounded host waits
// Host sync points (getters, forward with a loss, profile / timeline reads,
// model_free) of a model that talks to peers (NCCL or IPC) wait for a stream
// while polling NCCL's asynchronous error state: a failed or never-completing
// collective, or a peer that died, returns MGGCN_ENCCL (communicators
// aborted, model poisoned) instead of hanging the caller.  The wait limit is
// MGGCN_SYNC_TIMEOUT_S seconds (default 600).
static double sync_timeout_s() {
    static double t = -1;
    if (t < 0) {
        const char* e = getenv("MGGCN_SYNC_TIMEOUT_S");
        t = e ? atof(e) : 600.0;
        if (!(t > 0)) t = 600.0;
    }
    return t;
}

static void abort_comms(mggcn_model_s* m) {
    for (ncclComm_t* c : {&m->comm_bc, &m->comm_pair, &m->comm})
        if (*c) {
            ncclCommAbort(*c);
            *c = nullptr;
        }
}

static int poll_comm_errors(mggcn_model_s* m) {
    for (ncclComm_t c : {m->comm, m->comm_bc, m->comm_pair}) {
        if (!c) continue;
        ncclResult_t ae = ncclSuccess;
        const ncclResult_t r = ncclCommGetAsyncError(c, &ae);
        if (r != ncclSuccess || ae != ncclSuccess) {
            set_error(std::string("NCCL async error: ") + ncclGetErrorString(r != ncclSuccess ? r : ae));
            abort_comms(m);
            m->hung = true;
            return MGGCN_ENCCL;
        }
    }
    return MGGCN_OK;
}

static int sync_stream(mggcn_model_s* m, cudaStream_t s) {
    if (!m->comm && !m->ipc) {
        CK(cudaStreamSynchronize(s));
        return MGGCN_OK;
    }
    const auto t0 = std::chrono::steady_clock::now();
    for (;;) {
        const cudaError_t q = cudaStreamQuery(s);
        if (q == cudaSuccess) break;
        if (q != cudaErrorNotReady) {
            set_error(std::string("CUDA error while waiting: ") + cudaGetErrorString(q));
            return MGGCN_ECUDA;
        }
        RC(poll_comm_errors(m));
        const double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        if (el > sync_timeout_s()) {
            set_error("communication timeout: a stream waited more than MGGCN_SYNC_TIMEOUT_S s for peers "
                      "(collective or peer flag never completed)");
            abort_comms(m);
            m->hung = true;
            return MGGCN_ENCCL;
        }
        std::this_thread::sleep_for(std::chrono::microseconds(50));
    }
    return poll_comm_errors(m);
}

static int sync_both(mggcn_model_s* m) {
    RC(sync_stream(m, m->cs));
    return sync_stream(m, m->ms);
}

#define MODEL_GUARD(m)                                              \
    do {                                                            \
        if (!(m)) {                                                 \
            set_error("NULL model");                                \
            return MGGCN_EINVAL;                                    \
        }                                                           \
        if ((m)->poisoned) {                                        \
            set_error("model is poisoned by an earlier CUDA/NCCL error"); \
            return (m)->poisoned;                                   \
        }                                                           \
    } while (0)

// ------------------------------------------------------------- creation
static int model_init_common(mggcn_model_s* m, const mggcn_part* parts, int32_t nlocal, int32_t L,
                             const int32_t* dims, uint32_t flags) {
    if (!parts || nlocal < 1) {
        set_error("model: parts / nlocal invalid");
        return MGGCN_EINVAL;
    }
    RC(check_dims(L, dims));
    const mggcn_part_s* p0 = parts[0];
    if (!p0) {
        set_error("model: NULL part");
        return MGGCN_EINVAL;
    }
    m->P = p0->P;
    m->nlocal = nlocal;
    m->flags = flags;
    m->L = L;
    m->c = (flags & MGGCN_F_REPL2) ? 2 : 1;
    if ((flags & MGGCN_F_REPLICA1) && (m->c == 1 || nlocal != 1)) {
        set_error("model: MGGCN_F_REPLICA1 needs MGGCN_F_REPL2 and nlocal = 1");
        return MGGCN_EINVAL;
    }
    if (m->c > 1 && (m->P < 2 || m->P % m->c)) {
        set_error("model: MGGCN_F_REPL2 needs an even number P' >= 2 of row blocks");
        return MGGCN_EINVAL;
    }
    if (m->c > 1 && (flags & MGGCN_F_IPC)) {
        set_error("model: MGGCN_F_REPL2 is not implemented for MGGCN_F_IPC");
        return MGGCN_EUNSUPPORTED;
    }
    if (nlocal != 1 && nlocal != m->c * m->P) {
        set_error("model: nlocal must be 1 or P (loopback; 2P' with MGGCN_F_REPL2)");
        return MGGCN_EINVAL;
    }
    for (int i = 0; i < nlocal; ++i) {
        const mggcn_part_s* pi = parts[i];
        if (!pi || pi->P != m->P || pi->n != p0->n || pi->pattern != p0->pattern ||
            (nlocal > 1 && pi->rank != i % m->P) || pi->perm != p0->perm) {
            set_error("model: parts must come from the same graph / P / seed (and be ranks 0..P-1 in loopback)");
            return MGGCN_EINVAL;
        }
    }
    m->pattern = p0->pattern;
    m->d.assign(dims, dims + L + 1);
    m->ld.resize(L + 1);
    for (int l = 0; l <= L; ++l) m->ld[l] = ld_of(m->d[l]);
    m->order.resize(L);
    for (int l = 0; l < L; ++l) m->order[l] = m->d[l] < m->d[l + 1] ? S_ORDER : G_ORDER;   // §4.4, reading C10
    if (flags & MGGCN_F_CACHE_L0) m->order[0] = S_ORDER;   // T0 = Â'^T X is reused across epochs
    m->woff.resize(L);
    m->wtotal = 0;
    for (int l = 0; l < L; ++l) {
        m->woff[l] = m->wtotal;
        m->wtotal += round_up(m->d[l] * m->ld[l + 1], 64);
    }
    m->hw_ld = 4;
    m->bc_ld = 4;
    for (int l = 0; l < L; ++l) {
        if (m->order[l] == G_ORDER) {
            m->hw_ld = std::max(m->hw_ld, m->ld[l + 1]);
            m->bc_ld = std::max(m->bc_ld, m->ld[l + 1]);
        } else {
            m->bc_ld = std::max(m->bc_ld, m->ld[l]);
        }
    }
    m->max_rows_j = 0;
    for (int j = 0; j < m->P; ++j) m->max_rows_j = std::max(m->max_rows_j, p0->p[j + 1] - p0->p[j]);
    m->ranks.assign(nlocal, Rank());
    int64_t off = 0;
    for (int i = 0; i < nlocal; ++i) {
        Rank& r = m->ranks[i];
        r.part = parts[i];
        r.rank = parts[i]->rank;
        r.rep = nlocal > 1 ? i / m->P : ((flags & MGGCN_F_REPLICA1) ? 1 : 0);
        r.rows = parts[i]->nrows();
        r.row_off = off;
        off += r.rows;
        r.hF.assign(m->P, HostItems());
        r.hB.assign(m->P, HostItems());
        r.coalesced = !(flags & MGGCN_F_NO_COALESCE);
        if (r.coalesced) {
            r.cF.resize(m->P);
            for (int j = 0; j < m->P; ++j) coalesce(r.part->F[j], r.cF[j]);
            if (!r.part->shared_fb) {
                r.cB.resize(m->P);
                for (int j = 0; j < m->P; ++j) coalesce(r.part->B[j], r.cB[j]);
            }
        }
        std::vector<int32_t> order(r.rows);
        {
            const mggcn_part_s* pt = r.part;
            std::vector<int64_t> orig(r.rows);           // original id of local row rr
            const int64_t lo = pt->p[pt->rank];
            for (int64_t v = 0; v < pt->n; ++v) {
                const int64_t nv = pt->perm[v];
                if (nv >= lo && nv < lo + r.rows) orig[nv - lo] = v;
            }
            for (int64_t rr = 0; rr < r.rows; ++rr) order[rr] = (int32_t)rr;
            std::sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return orig[a] < orig[b]; });
        }
        for (int j = 0; j < m->P; ++j) {
            build_items(r.tF(j), r.hF[j], order);
            if (!r.part->shared_fb) build_items(r.tB(j), r.hB[j], order);
        }
        r.order_cache = order;
    }
    m->n_local = off;
    double e_row = 0;   // coalesced entries per row per remote tile (the compute / exchange regime)
    {
        double nnz = 0, rows = 0;
        for (auto& r : m->ranks)
            for (int j = 0; j < m->P; ++j)
                if (j != r.rank) {
                    nnz += (double)r.tF(j).rowptr.back();
                    rows += (double)r.rows;
                }
        e_row = rows > 0 ? nnz / rows : 0;
    }
    m->grp_b = choose_groups(m, e_row);
    if (m->grouped()) {
        const bool ipc = (flags & MGGCN_F_IPC) != 0;
        const int NG = n_groups(m);
        for (auto& r : m->ranks) {
            r.gF.assign(NG, HostTile());
            r.hgF.assign(NG, HostItems());
            if (!r.part->shared_fb) {
                r.gB.assign(NG, HostTile());
                r.hgB.assign(NG, HostItems());
            }
            for (int g = 0; g < NG; ++g) {
                std::vector<const HostTile*> tf, tb;
                for (int k = m->grp_b[g]; k < m->grp_b[g + 1]; ++k) {
                    const int j = remote_block(m, r.rank, k, ipc);
                    tf.push_back(&r.tF(j));
                    tb.push_back(&r.tB(j));
                }
                merge_group_tiles(tf, m->max_rows_j, r.gF[g]);
                build_items(r.gF[g], r.hgF[g], r.order_cache);
                if (!r.part->shared_fb) {
                    merge_group_tiles(tb, m->max_rows_j, r.gB[g]);
                    build_items(r.gB[g], r.hgB[g], r.order_cache);
                }
            }
        }
    }
    // Dense blocks of every launched tile (the local / per-stage tiles and the merged group
    // tiles); their work items are rebuilt over the residual entries.
    {
        const char* e = getenv("MGGCN_DENSE_THR");
        m->dense_thr = e ? atof(e) : kDenseThrDefault;
        const char* pe = getenv("MGGCN_DENSE_PIECES");
        m->dense_pieces = (pe && atoi(pe) == 2) ? 2 : 3;
        const char* fe = getenv("MGGCN_DENSE_MINFRAC");
        m->dense_min_frac = fe ? atof(fe) : kDenseMinFracDefault;
        const char* me = getenv("MGGCN_DENSE_MIN_ROWS");
        m->dense_min_rows = me ? atoll(me) : kDenseMinRowsDefault;
        const char* ne = getenv("MGGCN_DENSE_MIN_ENTRIES");
        m->dense_min_entries = ne ? atoll(ne) : kDenseMinEntriesDefault;
        if (!(m->dense_thr > 0) || (!m->ranks.empty() && !m->ranks[0].coalesced)) m->dense_thr = 0;
    }
    if (m->dense_thr > 0) {
        for (auto& r : m->ranks) {
            r.dF.assign(m->P, DenseHost());
            if (!r.part->shared_fb) r.dB.assign(m->P, DenseHost());
            for (int j = 0; j < m->P; ++j) {
                if (m->grouped() && j != r.rank) continue;
                plan_dense(r.tF(j), m->dense_thr, m->dense_min_frac, m->dense_min_rows, m->dense_min_entries, r.dF[j]);
                if (r.dF[j].active) {
                    r.hF[j] = HostItems();
                    build_items(r.lF(j), r.hF[j], r.order_cache);
                }
                if (!r.part->shared_fb) {
                    plan_dense(r.tB(j), m->dense_thr, m->dense_min_frac, m->dense_min_rows, m->dense_min_entries, r.dB[j]);
                    if (r.dB[j].active) {
                        r.hB[j] = HostItems();
                        build_items(r.lB(j), r.hB[j], r.order_cache);
                    }
                }
            }
            const int NG = n_groups(m);
            r.dgF.assign(NG, DenseHost());
            if (!r.part->shared_fb) r.dgB.assign(NG, DenseHost());
            for (int g = 0; g < NG; ++g) {
                plan_dense(r.gF[g], m->dense_thr, m->dense_min_frac, m->dense_min_rows, m->dense_min_entries, r.dgF[g]);
                if (r.dgF[g].active) {
                    r.hgF[g] = HostItems();
                    build_items(r.lgF(g), r.hgF[g], r.order_cache);
                }
                if (!r.part->shared_fb) {
                    plan_dense(r.gB[g], m->dense_thr, m->dense_min_frac, m->dense_min_rows, m->dense_min_entries, r.dgB[g]);
                    if (r.dgB[g].active) {
                        r.hgB[g] = HostItems();
                        build_items(r.lgB(g), r.hgB[g], r.order_cache);
                    }
                }
            }
        }
    }
    for (auto& r : m->ranks) std::vector<int32_t>().swap(r.order_cache);
    // the SpMM gathers address B with 32-bit float4 offsets: rows * ld/4 < 2^32
    if ((double)m->max_rows_j * (double)(std::max(m->bc_ld, m->ld[0]) / 4) >= 4294967296.0 ||
        (double)off * (double)(std::max(m->bc_ld, m->ld[0]) / 4) >= 4294967296.0) {
        set_error("model: a feature block exceeds 2^32 float4 (use more parts)");
        return MGGCN_EUNSUPPORTED;
    }
    // epoch work model, per this model's rows
    //   spmm_bytes   compulsory: 4 B per non-zero of the tile as partitioned (pattern-only; +4 B
    //                weighted) + rowptr + each gathered row once + each output row once
    //   struct bytes what the kernel's tile structure holds (coalesced entries: index +
    //                multiplicity value)
    auto spmm_work = [&](int dir, int64_t width) {
        for (auto& r : m->ranks)
            for (int j = 0; j < m->P; ++j) {
                if (!in_set(m, r.rep, j)) continue;      // 1.5D: the other replica's stages
                const HostTile& t = dir == 0 ? r.tF(j) : r.tB(j);
                const HostTile& raw = dir == 0 ? r.part->F[j] : r.part->tileB(j);
                const double nnz = (double)t.rowptr.back();
                const double nnz_raw = (double)raw.rowptr.back();
                const double rows_io = 4.0 * (double)width * (double)(t.ncols + t.nrows) + 4.0 * (double)(t.nrows + 1);
                m->w_spmm_bytes += nnz_raw * (raw.val.empty() ? 4.0 : 8.0) + rows_io;
                m->w_spmm_struct_bytes += nnz * (t.val.empty() ? 4.0 : 8.0) + rows_io;
                m->w_gather_bytes += nnz * 4.0 * (double)width;
                m->w_gather_raw_bytes += nnz_raw * 4.0 * (double)width;
                m->w_stages += 1.0;
                if (j != r.rank) m->w_bcast_bytes += 4.0 * (double)width * (double)t.ncols;
            }
    };
    int64_t root_rows = 0;                           // 1.5D: GEMM products only on the root replica
    for (auto& r : m->ranks)
        if (is_root(m, r)) root_rows += r.rows;
    for (int l = 0; l < L; ++l) {
        const int64_t w = m->order[l] == G_ORDER ? m->d[l + 1] : m->d[l];
        if (!(l == 0 && (flags & MGGCN_F_CACHE_L0))) spmm_work(0, w);   // steady state: T0 cached
        const double gf = 2.0 * (double)root_rows * (double)m->d[l] * (double)m->d[l + 1];
        const double dl = (double)m->d[l], dn = (double)m->d[l + 1];
        const double rows_fwd = m->order[l] == G_ORDER ? (double)root_rows : (double)m->n_local;
        m->w_gemm_flops += m->order[l] == G_ORDER ? gf : gf * (double)m->n_local / (double)std::max<int64_t>(root_rows, 1);
        m->w_gemm_bytes += 4.0 * (rows_fwd * (dl + dn) + dl * dn);            // F1: H W (or T0 W)
        m->w_gemm_flops += gf;                       // W_G
        m->w_gemm_bytes += 4.0 * ((double)root_rows * (dl + dn) + dl * dn);   // B2: H^T HW_G
        if (l > 0) {
            m->w_gemm_flops += gf;                   // H_G
            m->w_gemm_bytes += 4.0 * ((double)root_rows * (dl + 2.0 * dl + dn) + dl * dn);   // B3 + old-C mask
        }
        if (m->order[l] == G_ORDER) spmm_work(1, m->d[l + 1]);   // backward SpMM (Eq. 9)
    }
    m->w_ce_bytes = 2.0 * 4.0 * (double)root_rows * (double)m->d[L];
    return MGGCN_OK;
}

extern "C" int mggcn_workspace_bytes(const mggcn_part* parts, int32_t nlocal, int32_t L, const int32_t* dims,
                                     uint32_t flags, size_t* bytes) {
    if (!bytes) {
        set_error("workspace_bytes: NULL out");
        return MGGCN_EINVAL;
    }
    mggcn_model_s tmp;
    try {
        RC(model_init_common(&tmp, parts, nlocal, L, dims, flags));
    } catch (const std::bad_alloc&) {
        set_error("workspace_bytes: out of host memory");
        return MGGCN_ENOMEM;
    }
    Bump b;
    plan_buffers(&tmp, b);
    *bytes = b.off + 256;
    return MGGCN_OK;
}

extern "C" int mggcn_nccl_unique_id(void* out128) {
    if (!out128) {
        set_error("nccl_unique_id: NULL out");
        return MGGCN_EINVAL;
    }
    ncclUniqueId id;
    NK(ncclGetUniqueId(&id));
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
    std::memcpy(out128, &id, 128);
    return MGGCN_OK;
}

static void destroy(mggcn_model_s* m) {
    if (!m) return;
    // bounded: a model whose peers are gone must still be freeable (its comms are aborted)
    if (!m->hung && m->cs && m->ms && sync_both(m) != MGGCN_OK) m->hung = true;
    if (m->hung) {
        abort_comms(m);
        delete m;   // streams / events / graph of a hung model are left to process teardown
        return;
    }
    for (auto& r : m->ranks)
        for (int s = 0; s < 2; ++s) {
            if (r.ev_bc[s]) cudaEventDestroy(r.ev_bc[s]);
            if (r.ev_free[s]) cudaEventDestroy(r.ev_free[s]);
        }
    if (m->cp) cudaStreamSynchronize(m->cp);
    for (cudaEvent_t e : {m->ev_begin, m->ev_comm_end, m->ev_tmp, m->ev_wg, m->ev_comm_done, m->ev_pref, m->ev_xfree[0],
                          m->ev_xfree[1], m->ev_stage})
        if (e) cudaEventDestroy(e);
    for (auto& t : m->tl_recs) {
        cudaEventDestroy(t.a);
        cudaEventDestroy(t.b);
    }
    if (m->cp) cudaStreamDestroy(m->cp);
    for (auto& rec : m->prof_recs) {
        cudaEventDestroy(std::get<1>(rec));
        cudaEventDestroy(std::get<2>(rec));
    }
    for (auto e : m->prof_pool) cudaEventDestroy(e);
    if (m->ege) cudaGraphExecDestroy(m->ege);
    if (m->eg) cudaGraphDestroy(m->eg);
    if (m->comm_bc) ncclCommDestroy(m->comm_bc);
    if (m->comm_pair) ncclCommDestroy(m->comm_pair);
    if (m->comm) ncclCommDestroy(m->comm);
    for (void* p : m->ipc_opened)
        if (p) cudaIpcCloseMemHandle(p);
    delete m;
}

// Start-up check of a fresh NCCL communicator (and the 1.5D sub-communicators):
// one all-reduce of (rank + 1) and one broadcast of a known value from rank 0,
// verified on the host with a bounded wait, so a mis-wired job fails here with
// MGGCN_ENCCL instead of hanging or corrupting the first epoch.
static int nccl_selfcheck_one(mggcn_model_s* m, ncclComm_t c, float* buf, const char* what) {
    int nranks = 0, me = 0;
    NK(ncclCommCount(c, &nranks));
    NK(ncclCommUserRank(c, &me));
    const float init[2] = {(float)(me + 1), me == 0 ? 4242.0f : -1.0f};
    CK(cudaMemcpyAsync(buf, init, sizeof(init), cudaMemcpyHostToDevice, m->ms));
    NK(ncclGroupStart());
    NK(ncclAllReduce(buf, buf, 1, ncclFloat32, ncclSum, c, m->ms));
    NK(ncclBroadcast(buf + 1, buf + 1, 1, ncclFloat32, 0, c, m->ms));
    NK(ncclGroupEnd());
    float got[2] = {0, 0};
    CK(cudaMemcpyAsync(got, buf, sizeof(got), cudaMemcpyDeviceToHost, m->ms));
    RC(sync_stream(m, m->ms));
    const float want = 0.5f * (float)nranks * (float)(nranks + 1);
    if (got[0] != want || got[1] != 4242.0f) {
        set_error(std::string("model_create: NCCL self-check failed on the ") + what + " communicator (all-reduce " +
                  std::to_string(got[0]) + " != " + std::to_string(want) + " or broadcast " + std::to_string(got[1]) +
                  " != 4242)");
        return MGGCN_ENCCL;
    }
    return MGGCN_OK;
}

static int nccl_selfcheck(mggcn_model_s* m) {
    float* buf = nullptr;
    CK(cudaMalloc(&buf, 4 * sizeof(float)));
    int rc = nccl_selfcheck_one(m, m->comm, buf, "world");
    if (rc == MGGCN_OK && m->comm_bc) rc = nccl_selfcheck_one(m, m->comm_bc, buf, "replica-group");
    if (rc == MGGCN_OK && m->comm_pair) rc = nccl_selfcheck_one(m, m->comm_pair, buf, "row-block-pair");
    if (!m->hung) cudaFree(buf);
    return rc;
}

extern "C" int mggcn_model_create(const mggcn_part* parts, int32_t nlocal, int32_t L, const int32_t* dims,
                                  uint32_t flags, const void* nccl_id128, void* workspace, size_t ws_bytes,
                                  uintptr_t compute_stream, uintptr_t comm_stream, mggcn_model* out) {
    if (!out) {
        set_error("model_create: NULL out");
        return MGGCN_EINVAL;
    }
    *out = nullptr;
    mggcn_model_s* m = new (std::nothrow) mggcn_model_s();
    if (!m) {
        set_error("model_create: out of host memory");
        return MGGCN_ENOMEM;
    }
    int rc;
    try {
        rc = model_init_common(m, parts, nlocal, L, dims, flags);
    } catch (const std::bad_alloc&) {
        rc = MGGCN_ENOMEM;
        set_error("model_create: out of host memory");
    }
    if (rc != MGGCN_OK) {
        delete m;
        return rc;
    }
    m->ipc = (flags & MGGCN_F_IPC) && m->P > 1 && nlocal == 1;
    if ((flags & MGGCN_F_IPC) && (nlocal != 1 || nccl_id128)) {
        set_error("model_create: MGGCN_F_IPC needs nlocal = 1 and nccl_id128 = NULL");
        delete m;
        return MGGCN_EINVAL;
    }
    if (m->ipc && !ipc_stream_memops_available()) {
        set_error("model_create: MGGCN_F_IPC needs cuStreamWaitValue32 / cuStreamWriteValue32");
        delete m;
        return MGGCN_EUNSUPPORTED;
    }
    m->solo = m->P > 1 && nlocal == 1 && !nccl_id128 && !m->ipc && (flags & MGGCN_F_NO_BCAST) && m->c == 1;
    if (m->P > 1 && nlocal == 1 && !nccl_id128 && !m->ipc && !m->solo) {
        set_error("model_create: P > 1 with nlocal = 1 needs an NCCL unique id (or MGGCN_F_IPC, or the "
                  "MGGCN_F_NO_BCAST solo timing mode)");
        delete m;
        return MGGCN_EINVAL;
    }
    Bump sz;
    plan_buffers(m, sz);
    if (!workspace || (reinterpret_cast<uintptr_t>(workspace) & 255) || ws_bytes < sz.off + 256) {
        set_error("model_create: workspace NULL, misaligned (256 B) or smaller than mggcn_workspace_bytes");
        delete m;
        return MGGCN_EINVAL;
    }
    Bump b;
    b.base = static_cast<char*>(workspace);
    plan_buffers(m, b);
    m->ws_base = static_cast<char*>(workspace);
    m->ws_bytes = sz.off;
    m->cs = reinterpret_cast<cudaStream_t>(compute_stream);
    m->ms = reinterpret_cast<cudaStream_t>(comm_stream);
    auto fail = [&](int code) {
        destroy(m);
        return code;
    };
    if (cudaStreamCreateWithFlags(&m->cp, cudaStreamNonBlocking) != cudaSuccess) {
        set_error("model_create: cudaStreamCreate failed");
        return fail(MGGCN_ECUDA);
    }
    for (cudaEvent_t* e : {&m->ev_begin, &m->ev_comm_end, &m->ev_tmp, &m->ev_wg, &m->ev_comm_done, &m->ev_pref,
                           &m->ev_xfree[0], &m->ev_xfree[1], &m->ev_stage})
        if (cudaEventCreateWithFlags(e, cudaEventDisableTiming) != cudaSuccess) {
            set_error("model_create: cudaEventCreate failed");
            return fail(MGGCN_ECUDA);
        }
    for (auto& r : m->ranks)
        for (int s = 0; s < 2; ++s)
            if (cudaEventCreateWithFlags(&r.ev_bc[s], cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&r.ev_free[s], cudaEventDisableTiming) != cudaSuccess) {
                set_error("model_create: cudaEventCreate failed");
                return fail(MGGCN_ECUDA);
            }
    rc = upload_static(m);
    if (rc != MGGCN_OK) return fail(rc);
    rc = plan_gemms(m);
    if (rc != MGGCN_OK) return fail(rc);
    if (m->P > 1 && nlocal == 1 && !m->ipc && !m->solo) {
        ncclUniqueId id;
        std::memcpy(&id, nccl_id128, 128);
        ncclConfig_t cfg = NCCL_CONFIG_INITIALIZER;
        const char* mc = getenv("MGGCN_NCCL_MAX_CTAS");
        cfg.maxCTAs = mc ? atoi(mc) : 16;
        const Rank& r0 = m->ranks[0];
        ncclResult_t nr = ncclCommInitRankConfig(&m->comm, m->c * m->P, id, r0.rep * m->P + r0.rank, &cfg);
        if (nr != ncclSuccess) {
            set_error(std::string("model_create: ncclCommInitRankConfig: ") + ncclGetErrorString(nr));
            m->comm = nullptr;
            return fail(MGGCN_ENCCL);
        }
        if (m->c > 1) {   // 1.5D: replica group (broadcasts, rank = block index) and row-block pair
            nr = ncclCommSplit(m->comm, r0.rep, r0.rank, &m->comm_bc, &cfg);
            if (nr == ncclSuccess) nr = ncclCommSplit(m->comm, r0.rank, r0.rep, &m->comm_pair, &cfg);
            if (nr != ncclSuccess) {
                set_error(std::string("model_create: ncclCommSplit: ") + ncclGetErrorString(nr));
                return fail(MGGCN_ENCCL);
            }
        }
        rc = nccl_selfcheck(m);
        if (rc != MGGCN_OK) return fail(rc);
    }
    if (cudaStreamSynchronize(m->cs) != cudaSuccess) {
        set_error(std::string("model_create: ") + cudaGetErrorString(cudaGetLastError()));
        return fail(MGGCN_ECUDA);
    }
    *out = m;
    return MGGCN_OK;
}

extern "C" void mggcn_model_free(mggcn_model m) { destroy(m); }

// ------------------------------------------------------------------ IPC
// Blob layout (MGGCN_IPC_BLOB_BYTES = 128): cudaIpcMemHandle_t (64 B) of the
// allocation holding the workspace | uint64 offset of the workspace in it |
// int32 rank | int32 P | uint64 symmetric-region bytes | zero padding.
namespace {
struct IpcBlob {
    cudaIpcMemHandle_t h;
    uint64_t off;
    int32_t rank, P;
    uint64_t ws_bytes;
    char pad[128 - sizeof(cudaIpcMemHandle_t) - 24];
};
static_assert(sizeof(IpcBlob) == MGGCN_IPC_BLOB_BYTES, "IPC blob size");
}  // namespace

extern "C" int mggcn_ipc_export(mggcn_model m, void* blob) {
    MODEL_GUARD(m);
    if (!m->ipc || !blob) {
        set_error("ipc_export: model not created with MGGCN_F_IPC (P > 1), or NULL blob");
        return MGGCN_EINVAL;
    }
    void* base = nullptr;
    size_t size = 0;
    if (ipc_alloc_base(m->ws_base, &base, &size)) {
        set_error("ipc_export: cannot find the allocation holding the workspace");
        return MGGCN_ECUDA;
    }
    IpcBlob b{};
    if (cudaIpcGetMemHandle(&b.h, base) != cudaSuccess) {
        set_error(std::string("ipc_export: cudaIpcGetMemHandle: ") + cudaGetErrorString(cudaGetLastError()));
        return MGGCN_ECUDA;
    }
    b.off = (uint64_t)(m->ws_base - static_cast<char*>(base));
    b.rank = m->ranks[0].rank;
    b.P = m->P;
    b.ws_bytes = m->sym_bytes;
    std::memcpy(blob, &b, sizeof b);
    return MGGCN_OK;
}

extern "C" int mggcn_ipc_connect(mggcn_model m, const void* blobs) {
    MODEL_GUARD(m);
    if (!m->ipc || !blobs || m->ipc_connected) {
        set_error("ipc_connect: not an MGGCN_F_IPC model, NULL blobs, or already connected");
        return MGGCN_EINVAL;
    }
    const int P = m->P, me = m->ranks[0].rank;
    std::vector<IpcBlob> bl(P);
    std::memcpy(bl.data(), blobs, sizeof(IpcBlob) * P);
    for (int q = 0; q < P; ++q)
        if (bl[q].rank != q || bl[q].P != P || bl[q].ws_bytes != m->sym_bytes) {
            set_error("ipc_connect: blobs must be rank-ordered exports of models with the same P and plan");
            return MGGCN_EINVAL;
        }
    m->peer_ws.assign(P, nullptr);
    m->ipc_opened.assign(P, nullptr);
    for (int q = 0; q < P; ++q) {
        if (q == me) {
            m->peer_ws[q] = m->ws_base;
            continue;
        }
        void* p = nullptr;
        if (cudaIpcOpenMemHandle(&p, bl[q].h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
            set_error(std::string("ipc_connect: cudaIpcOpenMemHandle(rank ") + std::to_string(q) +
                      "): " + cudaGetErrorString(cudaGetLastError()));
            return MGGCN_ECUDA;
        }
        m->ipc_opened[q] = p;
        m->peer_ws[q] = static_cast<char*>(p) + bl[q].off;
    }
    m->ipc_connected = true;
    return MGGCN_OK;
}

// ---------------------------------------------------------------- weights
static int check_layer(mggcn_model_s* m, int32_t layer) {
    if (layer < 0 || layer >= m->L) {
        set_error("layer out of range");
        return MGGCN_EINVAL;
    }
    return MGGCN_OK;
}

extern "C" int mggcn_set_weights(mggcn_model m, int32_t layer, const float* W) {
    MODEL_GUARD(m);
    RC(check_layer(m, layer));
    if (!W) {
        set_error("set_weights: NULL W");
        return MGGCN_EINVAL;
    }
    const int64_t din = m->d[layer], dout = m->d[layer + 1], ld = m->ld[layer + 1];
    int rc = MGGCN_OK;
    auto body = [&]() -> int {
        CK(cudaMemcpy2DAsync(m->W + m->woff[layer], ld * 4, W, dout * 4, dout * 4, din, cudaMemcpyHostToDevice, m->cs));
        RC(refresh_weight_splits(m));
        CK(cudaMemsetAsync(m->Mom, 0, sizeof(float) * m->wtotal, m->cs));
        CK(cudaMemsetAsync(m->Vel, 0, sizeof(float) * m->wtotal, m->cs));
        RC(sync_stream(m, m->cs));
        return MGGCN_OK;
    };
    rc = body();
    m->t = 0;
    return poison(m, rc);
}

extern "C" int mggcn_get_weights(mggcn_model m, int32_t layer, float* W) {
    MODEL_GUARD(m);
    RC(check_layer(m, layer));
    const int64_t din = m->d[layer], dout = m->d[layer + 1], ld = m->ld[layer + 1];
    auto body = [&]() -> int {
        CK(cudaMemcpy2DAsync(W, dout * 4, m->W + m->woff[layer], ld * 4, dout * 4, din, cudaMemcpyDeviceToHost, m->cs));
        RC(sync_stream(m, m->cs));
        return MGGCN_OK;
    };
    return poison(m, body());
}

static int wait_wg(mggcn_model_s* m) {
    if (m->need_wg_wait) {
        CK(cudaStreamWaitEvent(m->cs, m->ev_wg, 0));
        m->need_wg_wait = false;
    }
    return MGGCN_OK;
}

extern "C" int mggcn_get_grad(mggcn_model m, int32_t layer, float* WG) {
    MODEL_GUARD(m);
    RC(check_layer(m, layer));
    const int64_t din = m->d[layer], dout = m->d[layer + 1], ld = m->ld[layer + 1];
    auto body = [&]() -> int {
        RC(wait_wg(m));
        CK(cudaMemcpy2DAsync(WG, dout * 4, m->WG + m->woff[layer], ld * 4, dout * 4, din, cudaMemcpyDeviceToHost, m->cs));
        RC(sync_stream(m, m->cs));
        return MGGCN_OK;
    };
    return poison(m, body());
}

extern "C" int mggcn_get_adam(mggcn_model m, int32_t layer, float* mom, float* vel, int64_t* t) {
    MODEL_GUARD(m);
    RC(check_layer(m, layer));
    const int64_t din = m->d[layer], dout = m->d[layer + 1], ld = m->ld[layer + 1];
    auto body = [&]() -> int {
        if (mom)
            CK(cudaMemcpy2DAsync(mom, dout * 4, m->Mom + m->woff[layer], ld * 4, dout * 4, din, cudaMemcpyDeviceToHost,
                                 m->cs));
        if (vel)
            CK(cudaMemcpy2DAsync(vel, dout * 4, m->Vel + m->woff[layer], ld * 4, dout * 4, din, cudaMemcpyDeviceToHost,
                                 m->cs));
        RC(sync_stream(m, m->cs));
        return MGGCN_OK;
    };
    if (t) *t = m->t;
    return poison(m, body());
}

extern "C" int mggcn_set_adam(mggcn_model m, int32_t layer, const float* mom, const float* vel, int64_t t) {
    MODEL_GUARD(m);
    RC(check_layer(m, layer));
    if (!mom || !vel || t < 0) {
        set_error("set_adam: NULL moments or t < 0");
        return MGGCN_EINVAL;
    }
    const int64_t din = m->d[layer], dout = m->d[layer + 1], ld = m->ld[layer + 1];
    auto body = [&]() -> int {
        CK(cudaMemcpy2DAsync(m->Mom + m->woff[layer], ld * 4, mom, dout * 4, dout * 4, din, cudaMemcpyHostToDevice,
                             m->cs));
        CK(cudaMemcpy2DAsync(m->Vel + m->woff[layer], ld * 4, vel, dout * 4, dout * 4, din, cudaMemcpyHostToDevice,
                             m->cs));
        RC(sync_stream(m, m->cs));
        return MGGCN_OK;
    };
    m->t = t;
    return poison(m, body());
}

// ---------------------------------------------------------------- forward
static int forward_impl(mggcn_model_s* m, const float* X, int64_t ldx, const int32_t* y, float* loss,
                        float* logits) {
    const int L = m->L;
    m->tl_nspmm = 0;
    // inputs -> internal buffers (this is the e2e H2D when X is host memory).
    // X == NULL: use the buffer filled by mggcn_prefetch on the copy stream.
    const bool use_cache = (m->flags & MGGCN_F_CACHE_L0) && m->t0_valid;
    if (!X) {
        CK(cudaStreamWaitEvent(m->cs, m->ev_pref, 0));
        RC(use_input_buffer(m, m->pref_buf));
        m->pref_buf = -1;
    } else {
        ProfScope ps(m, PC_OTHER, m->cs);
        if (use_cache) {
            // X is not read again (layer 0 starts from the cached T0): only the labels
            for (auto& r : m->ranks)
                if (r.rows) CK(cudaMemcpyAsync(r.y, y + r.row_off, sizeof(int32_t) * r.rows, cudaMemcpyDefault, m->cs));
        } else if (!m->ipc && device_zero_copy(m, X, ldx)) {
            // device X already in the padded layout: layer 0 reads it in place (it must stay
            // valid until this epoch's backward has run); labels are still copied
            RC(use_external_input(m, X));
            for (auto& r : m->ranks)
                if (r.rows) CK(cudaMemcpyAsync(r.y, y + r.row_off, sizeof(int32_t) * r.rows, cudaMemcpyDefault, m->cs));
        } else {
            RC(use_input_buffer(m, m->xcur));
            float* stage = m->ranks[0].HWB;   // free at this point of the epoch
            const int64_t stage_floats = m->ranks[0].rows * std::max<int64_t>(m->hw_ld, 4);
            RC(copy_inputs(m, m->xcur, X, ldx, y, m->cs, stage, stage_floats));
        }
    }
    for (int l = 0; l < L; ++l) {
        const bool relu_here = (l < L - 1) || (m->flags & MGGCN_F_RELU_LAST);
        int* layer_ids = m->layer_ids;
        layer_ids[l] = l;
        if (m->order[l] == G_ORDER) {
            for (auto& r : m->ranks)
                if (r.has_fwd[l] && is_root(m, r)) {
                    ProfScope ps(m, PC_GEMM, m->cs);
                    CK(gemm_launch(r.g_fwd[l], m->cs));                                  // Eq. 5 -> HWB (Eq. 16)
                }
            SpmmJob job{0, m->ld[l + 1], m->pattern, relu_here, src_HWB,
                        [](mggcn_model_s*, Rank& r, const void* c) { return r.AHWB[*static_cast<const int*>(c)]; },
                        &layer_ids[l]};
            RC(staged_spmm(m, job));                                                     // Eq. 6-7 -> AHWB (Eq. 17-18)
        } else {
            SpmmJob job{0, m->ld[0], m->pattern, false, src_X,
                        [](mggcn_model_s*, Rank& r, const void*) { return r.T0; }, nullptr};
            if (!use_cache) RC(staged_spmm(m, job));                                     // T = Â'^T X (§4.4)
            if (m->flags & MGGCN_F_CACHE_L0) m->t0_valid = true;
            for (auto& r : m->ranks)
                if (r.has_fwd[l]) {
                    ProfScope ps(m, PC_GEMM, m->cs);
                    CK(gemm_launch(r.g_fwd[l], m->cs));                                  // T W (+ReLU) -> AHWB_0
                }
        }
    }
    // ---- loss: |T|, logits out, fused CE fwd+bwd in place (Eq. 19)
    if (m->ipc && m->sc_seq) RC(ipc_wait_peers(m, m->cs, 5, m->sc_seq));   // peers read my last scalars
    for (auto& r : m->ranks) {
        CK(launch_count_labelled(r.y, r.rows, reinterpret_cast<int64_t*>(r.ce_partial), r.ntrain_local, m->cs));
        if (!is_root(m, r)) CK(cudaMemsetAsync(r.ntrain_local, 0, 8, m->cs));   // 1.5D: counted once (root)
    }
    RC(reduce_all(m, true));
    if (logits) {
        for (auto& r : m->ranks)
            if (r.rows)
                CK(cudaMemcpy2DAsync(logits + r.row_off * m->d[L], m->d[L] * 4, r.AHWB[L - 1], m->ld[L] * 4,
                                     m->d[L] * 4, r.rows, cudaMemcpyDeviceToDevice, m->cs));
    }
    const bool prescale = m->order[L - 1] == G_ORDER && m->pattern;
    for (auto& r : m->ranks) {
        ProfScope ps(m, PC_LOSS, m->cs);
        CK(launch_softmax_ce(r.AHWB[L - 1], r.rows, (int)m->d[L], m->ld[L], r.y, m->ntrain,
                             prescale ? r.inv_deg : nullptr, (m->flags & MGGCN_F_RELU_LAST) ? 1 : 0, r.ce_partial,
                             m->cs));
        CK(launch_sum_partials(r.ce_partial, kCeBlocks, r.loss_local, m->cs));
        if (!is_root(m, r)) CK(cudaMemsetAsync(r.loss_local, 0, 8, m->cs));
    }
    RC(reduce_all(m, false));
    if (loss) {
        double s = 0;
        int64_t nt = 0;
        CK(cudaMemcpyAsync(&s, m->loss_sum, 8, cudaMemcpyDeviceToHost, m->cs));
        CK(cudaMemcpyAsync(&nt, m->ntrain, 8, cudaMemcpyDeviceToHost, m->cs));
        RC(sync_stream(m, m->cs));
        *loss = (float)(s / (double)(nt > 0 ? nt : 1));
        if (m->comm) {
            ncclResult_t ae;
            if (ncclCommGetAsyncError(m->comm, &ae) == ncclSuccess && ae != ncclSuccess) {
                set_error(std::string("NCCL async error: ") + ncclGetErrorString(ae));
                return MGGCN_ENCCL;
            }
        }
    }
    return MGGCN_OK;
}

extern "C" int mggcn_forward(mggcn_model m, const float* X_local, int64_t ldx, const int32_t* y_local, float* loss,
                             float* logits_local) {
    NvtxRange nvtx_top("mggcn_forward");
    MODEL_GUARD(m);
    if (!X_local) {
        if (m->pref_buf < 0) {
            set_error("forward: X is NULL and no mggcn_prefetch is pending");
            return MGGCN_ESTATE;
        }
    } else if (!y_local || ldx < m->d[0]) {
        set_error("forward: NULL y or ldx < d_0");
        return MGGCN_EINVAL;
    }
    if (m->ipc && !m->ipc_connected) {
        set_error("forward: MGGCN_F_IPC model needs mggcn_ipc_connect first");
        return MGGCN_ESTATE;
    }
    RC(poison(m, wait_wg(m)));
    int rc = forward_impl(m, X_local, ldx, y_local, loss, logits_local);
    if (rc == MGGCN_OK && cudaEventRecord(m->ev_xfree[m->xcur], m->cs) != cudaSuccess) rc = MGGCN_ECUDA;
    if (rc == MGGCN_OK) m->state = ST_FWD;
    return poison(m, rc);
}

extern "C" int mggcn_prefetch(mggcn_model m, const float* X_local, int64_t ldx, const int32_t* y_local) {
    MODEL_GUARD(m);
    if (!X_local || !y_local || ldx < m->d[0]) {
        set_error("prefetch: NULL X/y or ldx < d_0");
        return MGGCN_EINVAL;
    }
    if (m->pref_buf >= 0) {
        set_error("prefetch: a prefetch is already pending (call mggcn_forward(X = NULL) first)");
        return MGGCN_ESTATE;
    }
    if (ipc_x_exchanged(m)) {
        set_error("prefetch: not with MGGCN_F_IPC and a SpMM-first layer 0 (peers read X from the "
                  "current input buffer, which must be the same on every rank)");
        return MGGCN_EUNSUPPORTED;
    }
    const int k = 1 - m->xcur;
    auto body = [&]() -> int {
        CK(cudaStreamWaitEvent(m->cp, m->ev_xfree[k], 0));   // last reader of buffer k is done
        RC(copy_inputs(m, k, X_local, ldx, y_local, m->cp, m->xstage, m->xstage_floats));
        CK(cudaEventRecord(m->ev_pref, m->cp));
        return MGGCN_OK;
    };
    int rc = body();
    if (rc == MGGCN_OK) m->pref_buf = k;
    return poison(m, rc);
}

extern "C" int mggcn_reset_cache(mggcn_model m) {
    MODEL_GUARD(m);
    m->t0_valid = false;
    return MGGCN_OK;
}

extern "C" int mggcn_get_loss(mggcn_model m, float* loss) {
    MODEL_GUARD(m);
    if (!loss) {
        set_error("get_loss: NULL out");
        return MGGCN_EINVAL;
    }
    double s = 0;
    int64_t nt = 0;
    auto body = [&]() -> int {
        CK(cudaMemcpyAsync(&s, m->loss_sum, 8, cudaMemcpyDeviceToHost, m->cs));
        CK(cudaMemcpyAsync(&nt, m->ntrain, 8, cudaMemcpyDeviceToHost, m->cs));
        RC(sync_stream(m, m->cs));
        return MGGCN_OK;
    };
    int rc = body();
    *loss = (float)(s / (double)(nt > 0 ? nt : 1));
    return poison(m, rc);
}

// --------------------------------------------------------------- backward
static int wgrad_reduce(mggcn_model_s* m, int l) {
    // per-rank partial W_G (Eq. 10) -> sum over ranks (reading C23)
    const int64_t din = m->d[l], dout = m->d[l + 1], ld = m->ld[l + 1];
    for (auto& r : m->ranks) {
        float* dst = (m->nlocal > 1 ? r.WG_local : m->ipc ? m->WGp : m->WG) + m->woff[l];
        if (m->ipc && m->wg_seq >= (uint32_t)m->L)
            RC(ipc_wait_peers(m, m->cs, 3, m->wg_seq + 1 - m->L));   // peers finished reading this slice
        if (r.has_wgrad[l] && is_root(m, r)) {   // 1.5D: the root replica contributes W_G (the other: zeros)
            {
                ProfScope ps(m, PC_GEMM, m->cs);
                CK(gemm_launch(r.g_wgrad[l], m->cs));
            }
            CK(launch_splitk_reduce(r.gemm_partial, r.g_wgrad[l].k_chunks, din, dout, dst, ld, m->cs));
        } else {
            CK(cudaMemsetAsync(dst, 0, sizeof(float) * din * ld, m->cs));
        }
    }
    if (m->nlocal > 1) {
        std::vector<const float*> in;
        for (auto& r : m->ranks) in.push_back(r.WG_local + m->woff[l]);
        ProfScope ps(m, PC_ALLRED, m->cs);
        CK(launch_sum_buffers(in.data(), (int)in.size(), m->WG + m->woff[l], din * ld, m->cs));
    } else if (m->ipc) {
        // W_G all-reduce as a pull-sum over peer memory, rank order (bitwise identical on all ranks)
        const uint32_t seq = ++m->wg_seq;
        RC(ipc_signal(m, m->cs, 2, seq));
        CK(cudaEventRecord(m->ev_tmp, m->cs));
        CK(cudaStreamWaitEvent(m->ms, m->ev_tmp, 0));
        {
            ProfScope ps(m, PC_ALLRED, m->ms);
            RC(ipc_wait_peers(m, m->ms, 2, seq));
            std::vector<const float*> in(m->P);
            for (int q = 0; q < m->P; ++q) in[q] = peer_ptr(m, q, m->WGp) + m->woff[l];
            CK(launch_sum_ranks_f32(in.data(), m->P, m->WG + m->woff[l], din * ld, m->ms));
        }
        RC(ipc_signal(m, m->ms, 3, seq));
        CK(cudaEventRecord(m->ev_wg, m->ms));
        m->need_wg_wait = true;
    } else if (m->comm) {
        CK(cudaEventRecord(m->ev_tmp, m->cs));
        CK(cudaStreamWaitEvent(m->ms, m->ev_tmp, 0));
        {
            ProfScope ps(m, PC_ALLRED, m->ms);
            NK(ncclAllReduce(m->WG + m->woff[l], m->WG + m->woff[l], (size_t)(din * ld), ncclFloat32, ncclSum, m->comm,
                             m->ms));
        }
        CK(cudaEventRecord(m->ev_wg, m->ms));
        m->need_wg_wait = true;
    }
    return MGGCN_OK;
}

static int backward_impl(mggcn_model_s* m) {
    const int L = m->L;
    int* layer_ids = m->layer_ids;
    for (int l = L - 1; l >= 0; --l) {
        layer_ids[l] = l;
        if (m->order[l] == G_ORDER) {
            // Eq. 9: HW_G = Â' · AHW_G (AHWB_l, pre-scaled by inv_deg when pattern-only) -> HWB (Eq. 20)
            SpmmJob job{1, m->ld[l + 1], false, false, src_AHWB,
                        [](mggcn_model_s*, Rank& r, const void*) { return r.HWB; }, &layer_ids[l]};
            RC(staged_spmm(m, job));
            RC(wgrad_reduce(m, l));                                           // Eq. 10
            if (l > 0)
                for (auto& r : m->ranks)
                    if (r.has_igrad[l] && is_root(m, r)) {
                        ProfScope ps(m, PC_GEMM, m->cs);
                        CK(gemm_launch(r.g_igrad[l], m->cs));                 // Eq. 11 + Eq. 8 mask -> AHWB_{l-1}
                    }
        } else {
            // S-order (l == 0 only): W_G = T^T Z_G; no input-feature gradient (§4.4 skip, reading C11)
            RC(wgrad_reduce(m, l));
        }
    }
    return MGGCN_OK;
}

extern "C" int mggcn_backward(mggcn_model m) {
    NvtxRange nvtx_top("mggcn_backward");
    MODEL_GUARD(m);
    if (m->state != ST_FWD) {
        set_error("backward: needs a preceding forward");
        return MGGCN_ESTATE;
    }
    int rc = backward_impl(m);
    if (rc == MGGCN_OK && cudaEventRecord(m->ev_xfree[m->xcur], m->cs) != cudaSuccess) rc = MGGCN_ECUDA;
    if (rc == MGGCN_OK) m->state = ST_BWD;
    return poison(m, rc);
}

static bool bad_hyper(float lr, float beta1, float beta2, float eps) {
    return !(lr > 0) || !(beta1 >= 0 && beta1 < 1) || !(beta2 >= 0 && beta2 < 1) || !(eps > 0);
}

static int step_impl(mggcn_model_s* m, float lr, float beta1, float beta2, float eps) {
    RC(wait_wg(m));
    m->t += 1;
    ProfScope ps(m, PC_ADAM, m->cs);
    CK(launch_adam(m->W, m->WG, m->Mom, m->Vel, m->wtotal, lr, beta1, beta2, eps, m->t, m->cs));
    RC(refresh_weight_splits(m));
    return MGGCN_OK;
}

extern "C" int mggcn_step(mggcn_model m, float lr, float beta1, float beta2, float eps) {
    NvtxRange nvtx_top("mggcn_step");
    MODEL_GUARD(m);
    if (int rc = poll_comm_errors(m)) return poison(m, rc);   // non-blocking
    if (m->state != ST_BWD) {
        set_error("step: needs a preceding backward");
        return MGGCN_ESTATE;
    }
    if (bad_hyper(lr, beta1, beta2, eps)) {
        set_error("step: bad hyper-parameters");
        return MGGCN_EINVAL;
    }
    int rc = step_impl(m, lr, beta1, beta2, eps);
    if (rc == MGGCN_OK) m->state = ST_READY;
    return poison(m, rc);
}

// ------------------------------------------------------- captured epochs
// The whole epoch (forward with no host loss read -> backward -> step) is
// captured once on the compute stream into a CUDA graph, with the comm stream
// forked and joined through the same events as the eager path; a replay is one
// cudaGraphLaunch, so the ~40 kernel launches of an epoch leave no host gaps.
// The graph bakes in every pointer (X, y, the workspace) and the launch plan;
// only Adam's step count changes between replays, and its node is re-set.
static void drop_epoch_graph(mggcn_model_s* m) {
    if (m->ege) cudaGraphExecDestroy(m->ege);
    if (m->eg) cudaGraphDestroy(m->eg);
    m->ege = nullptr;
    m->eg = nullptr;
    m->eg_adam = nullptr;
    m->eg_kernels = 0;
}

static bool is_device_ptr(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

extern "C" int mggcn_epoch_capture(mggcn_model m, const float* X_local, int64_t ldx, const int32_t* y_local, float lr,
                                   float beta1, float beta2, float eps) {
    MODEL_GUARD(m);
    if (!X_local || !y_local || ldx < m->d[0] || bad_hyper(lr, beta1, beta2, eps)) {
        set_error("epoch_capture: NULL X/y, ldx < d_0 or bad hyper-parameters");
        return MGGCN_EINVAL;
    }
    if (!is_device_ptr(X_local) || !is_device_ptr(y_local)) {
        set_error("epoch_capture: X and y must be device memory (the graph bakes in their addresses)");
        return MGGCN_EINVAL;
    }
    if (m->state != ST_READY || m->pref_buf >= 0) {
        set_error("epoch_capture: only between epochs, with no prefetch pending");
        return MGGCN_ESTATE;
    }
    if (m->ipc || (m->flags & MGGCN_F_CACHE_L0)) {
        set_error("epoch_capture: not with MGGCN_F_IPC (host-side sequence numbers) or MGGCN_F_CACHE_L0 "
                  "(first-epoch-only work)");
        return MGGCN_EUNSUPPORTED;
    }
    drop_epoch_graph(m);
    RC(poison(m, wait_wg(m)));
    const int64_t t_saved = m->t, launches0 = mggcn_kernel_launch_count();
    if (cudaStreamBeginCapture(m->cs, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
        set_error("epoch_capture: cudaStreamBeginCapture failed on the compute stream");
        cudaGetLastError();
        return MGGCN_EUNSUPPORTED;
    }
    m->capturing = true;
    int rc = forward_impl(m, X_local, ldx, y_local, nullptr, nullptr);
    if (rc == MGGCN_OK && cudaEventRecord(m->ev_xfree[m->xcur], m->cs) != cudaSuccess) rc = MGGCN_ECUDA;
    if (rc == MGGCN_OK) rc = backward_impl(m);
    if (rc == MGGCN_OK && cudaEventRecord(m->ev_xfree[m->xcur], m->cs) != cudaSuccess) rc = MGGCN_ECUDA;
    if (rc == MGGCN_OK) rc = step_impl(m, lr, beta1, beta2, eps);
    cudaGraph_t g = nullptr;
    const cudaError_t ec = cudaStreamEndCapture(m->cs, &g);
    m->capturing = false;
    m->t = t_saved;                 // nothing ran: the replays advance t
    m->state = ST_READY;
    m->need_wg_wait = false;        // the graph joins the comm stream back into the compute stream
    count_launches((int)(launches0 - mggcn_kernel_launch_count()));
    // events recorded during the capture became graph edges; re-record them on the
    // (no longer capturing) compute stream so that eager calls may wait on them again
    for (cudaEvent_t e : {m->ev_begin, m->ev_comm_end, m->ev_tmp, m->ev_wg, m->ev_comm_done, m->ev_xfree[0],
                          m->ev_xfree[1], m->ev_stage})
        if (e) cudaEventRecord(e, m->cs);
    for (auto& r : m->ranks)
        for (int k = 0; k < 2; ++k) {
            if (r.ev_bc[k]) cudaEventRecord(r.ev_bc[k], m->cs);
            if (r.ev_free[k]) cudaEventRecord(r.ev_free[k], m->cs);
        }
    if (rc != MGGCN_OK || ec != cudaSuccess || !g) {
        if (g) cudaGraphDestroy(g);
        cudaGetLastError();
        if (rc == MGGCN_OK) set_error(std::string("epoch_capture: ") + cudaGetErrorString(ec));
        return rc == MGGCN_ENCCL ? MGGCN_ENCCL : MGGCN_EUNSUPPORTED;
    }
    size_t nn = 0;
    cudaGraphGetNodes(g, nullptr, &nn);
    std::vector<cudaGraphNode_t> nodes(nn);
    if (nn) cudaGraphGetNodes(g, nodes.data(), &nn);
    for (cudaGraphNode_t nd : nodes) {
        cudaGraphNodeType ty;
        if (cudaGraphNodeGetType(nd, &ty) != cudaSuccess || ty != cudaGraphNodeTypeKernel) continue;
        ++m->eg_kernels;
        cudaKernelNodeParams kp;
        if (cudaGraphKernelNodeGetParams(nd, &kp) == cudaSuccess && kp.func == adam_kernel_func()) m->eg_adam = nd;
    }
    cudaGetLastError();
    m->eg = g;
    if (!m->eg_adam || cudaGraphInstantiate(&m->ege, g, 0) != cudaSuccess) {
        cudaGetLastError();
        drop_epoch_graph(m);
        set_error("epoch_capture: Adam node not found or cudaGraphInstantiate failed");
        return MGGCN_EUNSUPPORTED;
    }
    m->eg_lr = lr;
    m->eg_b1 = beta1;
    m->eg_b2 = beta2;
    m->eg_eps = eps;
    return MGGCN_OK;
}

extern "C" int mggcn_epoch_replay(mggcn_model m, int32_t epochs) {
    MODEL_GUARD(m);
    if (!m->ege) {
        set_error("epoch_replay: no captured epoch (mggcn_epoch_capture)");
        return MGGCN_ESTATE;
    }
    if (m->state != ST_READY || m->pref_buf >= 0 || epochs < 1) {
        set_error("epoch_replay: only between epochs, epochs >= 1");
        return m->state != ST_READY || m->pref_buf >= 0 ? MGGCN_ESTATE : MGGCN_EINVAL;
    }
    auto body = [&]() -> int {
        RC(wait_wg(m));
        for (int e = 0; e < epochs; ++e) {
            m->t += 1;
            CK(graph_set_adam(m->ege, m->eg_adam, m->W, m->WG, m->Mom, m->Vel, m->wtotal, m->eg_lr, m->eg_b1,
                              m->eg_b2, m->eg_eps, m->t));
            CK(cudaGraphLaunch(m->ege, m->cs));
            count_launches((int)m->eg_kernels);
        }
        // a later mggcn_prefetch refills an input buffer only after the replays
        for (cudaEvent_t e : m->ev_xfree) CK(cudaEventRecord(e, m->cs));
        return MGGCN_OK;
    };
    return poison(m, body());
}

// -------------------------------------------------------------- profiling
extern "C" int mggcn_get_profile(mggcn_model m, double* ms, int64_t* launches, int32_t reset) {
    MODEL_GUARD(m);
    if (int rc = sync_both(m)) return poison(m, rc);
    for (auto& rec : m->prof_recs) {
        float t = 0;
        cudaEventElapsedTime(&t, std::get<1>(rec), std::get<2>(rec));
        m->prof_ms[std::get<0>(rec)] += t;
        m->prof_n[std::get<0>(rec)] += 1;
        m->prof_pool.push_back(std::get<1>(rec));
        m->prof_pool.push_back(std::get<2>(rec));
    }
    m->prof_recs.clear();
    for (int c = 0; c < PC_N; ++c) {
        if (ms) ms[c] = m->prof_ms[c];
        if (launches) launches[c] = m->prof_n[c];
        if (reset) {
            m->prof_ms[c] = 0;
            m->prof_n[c] = 0;
        }
    }
    return MGGCN_OK;
}

extern "C" int mggcn_stage_groups(mggcn_model m, int32_t* sizes, int32_t cap) {
    MODEL_GUARD(m);
    const int ng = n_groups(m);
    for (int g = 0; g < ng && g < cap && sizes; ++g) sizes[g] = m->grp_b[g + 1] - m->grp_b[g];
    return ng;
}

extern "C" int mggcn_dense_stats(mggcn_model m, int64_t* out, int32_t n) {
    MODEL_GUARD(m);
    if (!out || n < 0) {
        set_error("dense_stats: bad arguments");
        return MGGCN_EINVAL;
    }
    // [0] blocks [1] entries in blocks [2] row groups [3] column chunks [4] entries of the launched
    // tiles (coalesced, blocks + residual), over every rank of this model and both directions
    int64_t v[5] = {0, 0, 0, 0, 0};
    for (auto& r : m->ranks) {
        for (const auto* dv : {&r.dF, &r.dB, &r.dgF, &r.dgB})
            for (const DenseHost& d : *dv)
                if (d.active) {
                    v[0] += d.n_tiles;
                    v[1] += d.nnz;
                    v[2] += d.n_groups;
                    v[3] += d.n_chunks;
                    v[4] += d.nnz;
                }
        for (int j = 0; j < m->P; ++j) {
            if (m->grouped() && j != r.rank) continue;
            v[4] += r.lF(j).rowptr.back();
            if (!r.part->shared_fb) v[4] += r.lB(j).rowptr.back();
        }
        for (int g = 0; g < n_groups(m); ++g) {
            v[4] += r.lgF(g).rowptr.back();
            if (!r.part->shared_fb) v[4] += r.lgB(g).rowptr.back();
        }
    }
    for (int i = 0; i < n && i < 5; ++i) out[i] = v[i];
    return 5;
}

extern "C" int mggcn_debug_poison(mggcn_model m, int32_t on) {
    MODEL_GUARD(m);
    if (on < 0 || on > 2) {
        set_error("debug_poison: on must be 0, 1 or 2");
        return MGGCN_EINVAL;
    }
    m->poison_bc = on != 0;
    m->break_bc_wait = on == 2;
    return MGGCN_OK;
}

extern "C" int mggcn_timeline_enable(mggcn_model m, int32_t on) {
    MODEL_GUARD(m);
    if (m->capturing) {
        set_error("timeline_enable: not during an epoch capture");
        return MGGCN_ESTATE;
    }
    if (on) m->flags |= MGGCN_F_TIMELINE;
    else m->flags &= ~(uint32_t)MGGCN_F_TIMELINE;
    return MGGCN_OK;
}

extern "C" int mggcn_get_timeline(mggcn_model m, int64_t cap, int32_t* meta, double* t_ms, int64_t* count,
                                  int32_t reset) {
    MODEL_GUARD(m);
    if (cap < 0 || (cap > 0 && (!meta || !t_ms))) {
        set_error("get_timeline: cap < 0 or NULL arrays");
        return MGGCN_EINVAL;
    }
    if (int rc = sync_both(m)) return poison(m, rc);
    const int64_t n = (int64_t)m->tl_recs.size();
    if (count) *count = n;
    for (int64_t i = 0; i < n && i < cap; ++i) {
        const auto& t = m->tl_recs[i];
        for (int k = 0; k < 5; ++k) meta[5 * i + k] = t.meta[k];
        float a = 0, b = 0;
        cudaEventElapsedTime(&a, m->tl_recs[0].a, t.a);
        cudaEventElapsedTime(&b, m->tl_recs[0].a, t.b);
        t_ms[2 * i] = a;
        t_ms[2 * i + 1] = b;
    }
    if (reset) {
        for (auto& t : m->tl_recs) {
            m->prof_pool.push_back(t.a);
            m->prof_pool.push_back(t.b);
        }
        m->tl_recs.clear();
    }
    return MGGCN_OK;
}

extern "C" int mggcn_epoch_work_detail(mggcn_model m, double* out, int32_t n) {
    MODEL_GUARD(m);
    if (!out || n < 0) {
        set_error("epoch_work_detail: NULL out or n < 0");
        return MGGCN_EINVAL;
    }
    const double v[] = {m->w_spmm_bytes, m->w_spmm_struct_bytes, m->w_gather_bytes, m->w_gather_raw_bytes,
                        m->w_gemm_flops, m->w_gemm_bytes, m->w_bcast_bytes, m->w_ce_bytes, m->w_stages};
    const int32_t k = (int32_t)(sizeof(v) / sizeof(v[0]));
    for (int32_t i = 0; i < n && i < k; ++i) out[i] = v[i];
    return k;
}

extern "C" int mggcn_epoch_work(mggcn_model m, double* spmm_bytes, double* gather, double* flops, double* bcast) {
    if (!m) {
        set_error("NULL model");
        return MGGCN_EINVAL;
    }
    if (spmm_bytes) *spmm_bytes = m->w_spmm_bytes;   // SURVEY §8(d) compulsory (raw pattern)
    if (gather) *gather = m->w_gather_bytes;
    if (flops) *flops = m->w_gemm_flops;
    if (bcast) *bcast = m->w_bcast_bytes;
    return MGGCN_OK;
}

// ------------------------------------------------------------- test hooks
extern "C" int mggcn_debug_comm_delay(mggcn_model m, uint64_t seed, int32_t max_us) {
    MODEL_GUARD(m);
    if (max_us < 0 || max_us > 10000) {
        set_error("debug_comm_delay: max_us must be in [0, 10000]");
        return MGGCN_EINVAL;
    }
    m->delay_seed = seed;
    m->delay_ctr = 0;
    m->delay_max_us = max_us;
    return MGGCN_OK;
}

extern "C" int mggcn_debug_layer(mggcn_model m, int32_t layer, float* dst, int64_t ld) {
    MODEL_GUARD(m);
    RC(check_layer(m, layer));
    const int64_t w = m->d[layer + 1];
    if (!dst || ld < w) {
        set_error("debug_layer: NULL dst or ld < d_{l+1}");
        return MGGCN_EINVAL;
    }
    auto body = [&]() -> int {
        for (auto& r : m->ranks)
            if (r.rows)
                CK(cudaMemcpy2DAsync(dst + r.row_off * ld, ld * 4, r.AHWB[layer],
                                     m->ld[layer + 1] * 4, w * 4, r.rows, cudaMemcpyDefault, m->cs));
        RC(sync_stream(m, m->cs));
        return MGGCN_OK;
    };
    return poison(m, body());
}

extern "C" int mggcn_debug_spmm(mggcn_model m, int32_t dir, const float* B, int64_t ldb, int32_t width, float* out,
                                int64_t ldo) {
    MODEL_GUARD(m);
    if ((dir != 0 && dir != 1) || !B || !out || width <= 0 || (ldb & 3) || (ldo & 3) || ldb < width || ldo < width) {
        set_error("debug_spmm: bad arguments");
        return MGGCN_EINVAL;
    }
    if (m->P > 1 && m->nlocal == 1 && !m->solo) {
        set_error("debug_spmm: needs P == 1, loopback or the SOLO timing mode");
        return MGGCN_EUNSUPPORTED;
    }
    const int64_t w = round_up(width, 4);
    if (w > m->bc_ld && m->P > 1) {
        set_error("debug_spmm: width exceeds the model's broadcast buffers");
        return MGGCN_EINVAL;
    }
    // staging: per rank a contiguous (rows x w) input (pre-scaled by inv_deg for the
    // pattern-only backward) and output, carved from one cudaMalloc
    size_t tot = 0;
    for (auto& r : m->ranks) tot += 2 * (size_t)r.rows * w;
    float* scratch = nullptr;
    auto body = [&]() -> int {
        CK(cudaMalloc(&scratch, sizeof(float) * (tot + 64)));
        CK(cudaMemsetAsync(scratch, 0, sizeof(float) * (tot + 64), m->cs));
        struct Ctx {
            std::vector<float*> in, out;
        } ctx;
        size_t off = 0;
        for (auto& r : m->ranks) {
            ctx.in.push_back(scratch + off);
            off += (size_t)r.rows * w;
            ctx.out.push_back(scratch + off);
            off += (size_t)r.rows * w;
            const bool pre = dir == 1 && m->pattern;
            if (r.rows)
                CK(launch_scale_rows(B + r.row_off * ldb, ldb, ctx.in.back(), w, r.rows, width,
                                     pre ? r.inv_deg : nullptr, m->cs));
        }
        SpmmJob job{dir, w, dir == 0 && m->pattern, false,
                    [](mggcn_model_s* mm, Rank& r, const void* c) {
                        return static_cast<const Ctx*>(c)->in[&r - mm->ranks.data()];
                    },
                    [](mggcn_model_s* mm, Rank& r, const void* c) {
                        return static_cast<const Ctx*>(c)->out[&r - mm->ranks.data()];
                    },
                    &ctx};
        RC(staged_spmm(m, job));
        for (size_t i = 0; i < m->ranks.size(); ++i) {
            Rank& r = m->ranks[i];
            if (r.rows)
                CK(cudaMemcpy2DAsync(out + r.row_off * ldo, ldo * 4, ctx.out[i], w * 4, width * 4, r.rows,
                                     cudaMemcpyDeviceToDevice, m->cs));
        }
        RC(sync_stream(m, m->cs));
        return MGGCN_OK;
    };
    int rc = body();
    if (scratch) cudaFree(scratch);
    return poison(m, rc);
}

extern "C" int mggcn_debug_gemm(int32_t op, int64_t M, int64_t N, int64_t K, const float* A, int64_t lda,
                                const float* B, int64_t ldb, float* C, int64_t ldc, uint32_t flags, uintptr_t stream) {
    if (op < 0 || op > 2 || !A || !B || !C || ldc < N || M <= 0 || N <= 0 || K <= 0) {
        set_error("debug_gemm: bad arguments");
        return MGGCN_EINVAL;
    }
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const int gf = (flags & MGGCN_F_TF32X1) ? GEMM_TF32X1 : 0;
    float* scratch = nullptr;
    auto body = [&]() -> int {
        GemmPlan g;
        if (op == 2) {
            size_t pf = 0;
            if (gemm_plan_wgrad(g, M, N, K, A, lda, B, ldb, gf, &pf)) {
                set_error("debug_gemm: plan failed (alignment: pointers 16 B, lda/ldb multiple of 4; needs sm_100)");
                return MGGCN_EINVAL;
            }
            CK(cudaMalloc(&scratch, sizeof(float) * (pf + 4)));
            g.partial = scratch;
            CK(gemm_launch(g, s));
            CK(launch_splitk_reduce(scratch, g.k_chunks, M, N, C, ldc, s));
        } else {
            // B^T operand as K-major [N x K] hi / lo (op 0: transpose of B [K x N]; op 1: B [N x K] itself)
            const int64_t ldk = op == 0 ? round_up(K, 4) : ldb;
            CK(cudaMalloc(&scratch, sizeof(float) * (2 * N * ldk + 8)));
            float* bh = scratch;
            float* bl = scratch + N * ldk;
            CK(cudaMemsetAsync(scratch, 0, sizeof(float) * 2 * N * ldk, s));
            if (op == 0) CK(launch_split_weights(B, K, N, ldb, bh, bl, ldk, nullptr, nullptr, gf ? 1 : 0, s));
            else CK(launch_split_weights(B, N, K, ldb, nullptr, nullptr, 0, bh, bl, gf ? 1 : 0, s));
            if (gemm_plan_rows(g, M, N, K, A, lda, bh, bl, ldk, C, ldc, gf)) {
                set_error("debug_gemm: plan failed (alignment: pointers 16 B, lda/ldb multiple of 4; needs sm_100)");
                return MGGCN_EINVAL;
            }
            CK(gemm_launch(g, s));
        }
        CK(cudaStreamSynchronize(s));
        return MGGCN_OK;
    };
    int rc = body();
    if (scratch) cudaFree(scratch);
    return rc;
}
