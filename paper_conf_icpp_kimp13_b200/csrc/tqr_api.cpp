// tqr_api.cpp -- C ABI (include/tqr.h), plan/partition, tile-DAG scheduler on CUDA streams.
//
// Partition (Sec. IV.C): column tiles are owned per the distribution guide array,
// owner(j) = guide[j % len] (Eq. 12; reading Q13: every column, owner-computes).
// Tiles of an owned column are contiguous in the owner's HBM (tile (i, j) is nb x nb
// column-major), so panel k's reflectors (tiles k..p-1), T factors and explicit V are three
// contiguous ranges that are broadcast without packing.
//
// Schedule (Fig. 3 DAG; Sec. IV.D progress P:L1028-1039, re-designed): per step k
//   owner(k), panel stream : PANEL(k) = GEQRT(k,k) + TSQRT(k+1..p-1, k)       -> ev_panel[k]
//   every other owner d    : comm stream receives panel k (peer copy or ncclBroadcast)
//   owner(k+1), panel str. : lookahead UPDATE(k, column k+1) (waits rest(k-1))   -> ev_look[k]
//   every owner d, S update streams: UPDATE(k, its columns > k except the lookahead one),
//                            column lc on stream lc % S                          -> ev_u[u][k]
// so PANEL(k+1) overlaps the bulk trailing update of step k, and step k+1's updates of one
// stream start while other streams still finish step k (no wave-quantisation tail per step).
// The panel stream has the highest stream priority so freed SMs go to the critical path first.
#include "../../include/tqr.h"

#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <chrono>
#include <new>
#include <thread>
#include <numeric>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "nccl_dl.h"
#include "tqr_internal.h"

using tqr::PanelArgs;
using tqr::UpdateArgs;

namespace {

thread_local std::string g_create_error;

// NVTX ranges (header-only NVTX v3: free when no profiler is attached) around the ABI phases and
// every factorization step, so an nsys / ncu timeline shows load, PANEL(k) / BCAST(k) / UPDATE(k),
// R out, apply and solve.
struct NvtxRange {
    explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
    NvtxRange(const char* fmt, int k) {
        char b[48];
        snprintf(b, sizeof(b), fmt, k);
        nvtxRangePushA(b);
    }
    ~NvtxRange() { nvtxRangePop(); }
};

struct Owner {
    int id = 0;
    int dev = 0;
    std::vector<int32_t> cols;      // global column tiles owned (ascending)
    std::vector<int32_t> lidx;      // global j -> local index or -1
    int32_t* cols_dev = nullptr;
    // element type = the plan's dtype (double or float); sizes in elements
    void* tiles = nullptr;          // ncols * p * nb*nb
    void* T = nullptr;              // ncols * p * ib*nb
    void* Vimg = nullptr;           // ncols * p * vt     stage images of the reflector tiles (update-kernel operand)
    void* Vexp = nullptr;           // ncols * vt         stage image of the explicit V of each diagonal tile
    void* rb_tiles[2] = {nullptr, nullptr};
    void* rb_T[2] = {nullptr, nullptr};
    void* rb_V[2] = {nullptr, nullptr};
    unsigned* flags = nullptr;      // p * (nb/ib) * 5 panel-kernel publication flags
    unsigned* mflags = nullptr;     // tree mode: the merge chain's own flags (the domain jobs of the
                                    // same step stamp the main flags with the same epoch)
    void* io = nullptr;             // m x (nb*ncols) column-major mirror for host / remote I/O
    // tree mode (TS domains + flat TT merge chain, NEXT-1): per owned column, Dmax merge slots
    void* Mimg = nullptr;           // ncols * Dmax * vt   stage images of the merge reflectors (slot e)
    void* MT = nullptr;             // ncols * Dmax * ib*nb  merge T factors
    double* Mt = nullptr;           // Dmax * nb*nb        merge bottoms triu(R_e) -> V2 (factor scratch)
    void* rb_M[2] = {nullptr, nullptr};
    void* rb_MT[2] = {nullptr, nullptr};
    // FP32 plans: FP64 scratch of one panel column (the panel is factored in FP64, then narrowed)
    double* sc_col = nullptr;       // p * nb*nb
    double* sc_T = nullptr;         // p * ib*nb
    double* sc_Vimg = nullptr;      // p * nb*nb
    double* sc_Vexp = nullptr;      // nb*nb
    cudaStream_t s_panel = nullptr, s_upd = nullptr, s_comm = nullptr;
    cudaStream_t s_io = nullptr;                    // streamed tqr_factor: per-column H2D + a1, a8 + D2H
    cudaStream_t s_look = nullptr;                  // lookahead update overlapped with its own panel
    std::vector<cudaEvent_t> ev_load;               // ev_load[lc]: local column lc resident in tile layout
    std::vector<cudaEvent_t> ev_chunk, ev_dom;      // streamed tall factor: row chunk c loaded / its domains done
    std::vector<cudaStream_t> s_u;                  // bulk-update streams (column lc -> s_u[lc % S])
    std::vector<cudaEvent_t> ev_panel, ev_recv, ev_look;
    std::vector<cudaEvent_t> ev_prepanel;           // before PANEL(k)'s launch (remote trailing lookahead)
    unsigned long long* cflg = nullptr;             // remote trailing: chunk flags, 2 slots x kMaxChunks
    std::vector<std::vector<cudaEvent_t>> ev_u;     // ev_u[u][k]: stream u finished its step-k updates
    std::vector<std::vector<cudaEvent_t>> tm0, tm1; // profiling pairs per (u, k)
    std::vector<cudaEvent_t> tp0, tp1, tref;        // panel pairs, reference
    std::vector<cudaEvent_t> tb0, tb1;              // transfer pairs per step (stats[3])
    cudaEvent_t tl[4] = {nullptr, nullptr, nullptr, nullptr};   // layout pairs: load, store (stats[2])
    std::vector<std::vector<char>> tm_used;
    std::vector<char> tp_used, tb_used;
};

struct KStat {
    int64_t count = 0;
    double ms = 0.0, flops = 0.0;
};

// ---- CUDA-IPC transport (tqr_options.transport = TQR_TRANSPORT_IPC)
// Export blob of one rank: IPC handles of the allocations peers touch.
enum IpcSlot {
    H_FLAGS = 0,
    H_RB = 1,        // receive slots: H_RB + 5*s + {tiles, T, V, M, MT}
    H_TILES = 11, H_VIMG, H_T, H_VEXP, H_MIMG, H_MT,   // reflector storage (apply/solve replication)
    H_RSSEND,        // row split: this rank's R_g for the stage-2 gather
    kNH
};
struct IpcBlob {
    uint32_t magic;
    int32_t rank, dev, world;
    uint64_t present;            // bit i: handle i exported
    unsigned char uuid[16];      // the GPU's UUID (ordinals differ between processes)
    cudaIpcMemHandle_t h[kNH];
};
constexpr uint32_t kIpcMagic = 0x54515231u;   // "TQR1"
// 64-bit flags in each rank's flag block (waits are always on the waiter's own block):
constexpr int F_READY = 0;       // [slot]            panel of step k landed in my receive slot k%2 (root writes)
constexpr int F_FREED = 8;       // [2*src + slot]    rank src's slot is free for step k (src writes into root's block)
constexpr int F_DONE = 160;      // [src]             rank src finished factorization #E (its storage is final)
constexpr int F_APPLIED = 224;   // [src]             rank src finished apply/solve call #seq (its pulls)
constexpr int F_RSREADY = 288;   // [src]             row split: rank src's R_g is in its rs_send (rank 0's block)
constexpr int F_PULLED = 352;    //                   row split: rank 0 has pulled my R_g of #E (my block)
constexpr int F_CHUNK = 384;     // [slot*64 + c]     remote trailing: chunk c of the panel in my slot (root writes)
constexpr int kMaxChunks = 64;
constexpr int kFlagWords = 512;
constexpr int kIpcMaxWorld = 64;
struct IpcPeer {
    int dev = -1;
    unsigned char uuid[16] = {0};
    uint64_t* flags = nullptr;
    void* rb[2][5] = {{nullptr}};   // receive slot s: tiles, T, V, M, MT
    void* st[6] = {nullptr};        // tiles, Vimg, T, Vexp, Mimg, MT
    void* rs_send = nullptr;
};

}  // namespace

struct tqr_plan_s {
    int64_t m = 0, n = 0;
    int nb = 0, ib = 0, p = 0, q = 0;
    tqr_dtype dtype = TQR_F64;
    int es = 8;                     // element size in bytes
    int64_t vt = 0;                 // elements of one reflector-tile stage image (F64: nb*nb)
    int ndev = 1;
    std::vector<int32_t> guide;
    std::vector<int32_t> owner_of;  // size q
    bool logical = false;
    int rank = 0, world = 1;
    bool lookahead = true, profile = false;
    int nstreams = 4;               // bulk-update streams per owner (TQR_UPDATE_STREAMS), column lc -> lc % S
    int nstreams_io = 8;            // streamed factor: contiguous column chunks, one stream each
    int nstreams_alloc() const { return std::max(nstreams, nstreams_io); }
    int panel_split = 1;            // sub-slice CTAs per ib column block in the panel kernel
    int w_look = 0;                 // lookahead slice width (0 = default: 8 at nb >= 256, else 16)
    int tree_L = 0;                 // TS-domain length (tiles); 0 = flat TS chain
    int dmax = 1;                   // max domains of any step = ceil(p / tree_L)
    int tree_G = 0;                 // merge tree: groups of G heads per level (0 = one flat merge chain)
    int merge_split = 1;            // panel sub-slice split of the level-1 merge jobs
    // streamed tqr_factor (caller A not on the owner's device): column loads overlap the
    // factorization (panel k / the step-0 update of column j wait for ev_load), R of column k is
    // written back on s_io as soon as PANEL(k) completes
    void* prog = nullptr;           // wavefront apply progress flags (q * nslices)
    size_t prog_n = 0;
    bool la_overlap = true;         // FP64 flat lookahead runs beside PANEL(k) on per-tile flags
    bool w16 = true;                // FP64 bulk Q^T chains on 16 warps per CTA (TQR_W16=0: 8 warps)
    bool la_fits = true;            // ... only when its spinning CTAs leave SMs for the whole panel grid
    bool la_remote = false;         // the lookahead of column k+1 on ANOTHER owner trails PANEL(k) chunk by chunk
    int la_chunk = 8;               // tiles per trailing transfer chunk
    bool streamed = false;
    bool domains_done = false;      // streamed tall factor: the TS domains were launched per row chunk
    bool cp_probe = false;          // TQR_CRITICAL_PATH_PROBE=1 (diagnostic, wrong results): skip the
                                    // bulk updates -> panels + lookahead only = the critical path
    void* sA = nullptr;
    int64_t slda = 0;
    // merge tree of D domain heads: level l merges, in groups of G consecutive heads of stride G^l,
    // heads gG+1..gG+G-1 into head gG (one multi-job launch per level); G >= D: one flat chain
    int merge_group(int D) const { return tree_G > 1 ? tree_G : std::max(2, D); }
    int ndom(int k) const { return tree_L > 0 ? (p - k + tree_L - 1) / tree_L : 1; }
    bool tree_one_cta = true;       // domain phase: one CTA per domain (long domains) or wavefront jobs
    int tree_split = 1;             // panel split of the wavefront domain jobs
    std::vector<Owner> owners;      // in-process: ndev entries; multi-process: 1 (this rank)
    const tqr::NcclApi* nccl = nullptr;
    ncclComm_t comm = nullptr;
    bool factored = false, poisoned = false;
    unsigned epoch = 1;
    std::string err;
    KStat stats[4];
    int64_t launches = 0;
    // apply / solve workspace (single-device plans)
    void* bw = nullptr;
    size_t bw_elems = 0;
    int64_t* dflag = nullptr;

    // row split (tqr_options.row_split): per local owner a plan over its contiguous row block
    // (kids), a stage-2 plan on owner 0 (top) factoring the stacked triu(R_g) (stk, G*nb x n)
    bool rs = false;
    std::vector<tqr_plan> kids;
    std::vector<int> kid_owner, kid_dev;
    std::vector<int64_t> rs_r0, rs_rows;    // per owner id
    std::vector<void*> rs_zero;             // per kid: n x n zeros on its device
    tqr_plan top = nullptr;
    int top_dev = 0;
    void* stk = nullptr;
    void* rs_send = nullptr;
    void* rs_recv = nullptr;
    cudaStream_t rs_stream = nullptr;       // this process's gather stream

    bool nccl_mode = false;         // one process per GPU, panels broadcast with NCCL
    bool ipc_mode = false;          // one process per owner, panels copied into CUDA-IPC-mapped slots
    bool ipc_connected = false;
    uint64_t* flags64 = nullptr;    // this rank's IPC flag block (kFlagWords)
    std::vector<IpcPeer> peers;     // IPC: world entries (own entry = local pointers)
    std::vector<void*> ipc_opened;  // peer mappings to close
    uint64_t apply_seq = 0;         // IPC apply/solve collectives so far
    uint64_t fact_id = 0;           // flag value of the last completed factorization
    uint64_t rs_epoch = 0;          // row split factorizations so far
    // multi-owner apply / solve: single-owner replica of the factorization on this device
    tqr_plan rep = nullptr;
    uint64_t fact_gen = 0, rep_gen = 0;
    // issued-op trace of the last tqr_factor_tiles (tqr_issued_ops)
    std::vector<int32_t> issued;
    bool multiproc() const { return nccl_mode || ipc_mode; }
    bool f32() const { return dtype == TQR_F32; }
    // p + e elements
    template <class E = void>
    E* at(void* ptr, int64_t e) const { return reinterpret_cast<E*>(static_cast<char*>(ptr) + e * es); }
    Owner* local(int d) {
        if (multiproc()) return (d == rank) ? &owners[0] : nullptr;
        return &owners[d];
    }
};

namespace {

tqr_status fail(tqr_plan h, tqr_status st, const char* fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof(buf), fmt, ap);
    va_end(ap);
    if (h) {
        h->err = buf;
        if (st == TQR_ERR_CUDA || st == TQR_ERR_NCCL) h->poisoned = true;
    } else {
        g_create_error = buf;
    }
    return st;
}

#define CUDA_TRY(h, call)                                                                          \
    do {                                                                                           \
        cudaError_t e_ = (call);                                                                   \
        if (e_ != cudaSuccess)                                                                     \
            return fail((h), TQR_ERR_CUDA, "%s:%d %s -> %s", __FILE__, __LINE__, #call,            \
                        cudaGetErrorString(e_));                                                   \
    } while (0)

#define NCCL_TRY(h, call)                                                                          \
    do {                                                                                           \
        ncclResult_t r_ = (call);                                                                  \
        if (r_ != ncclSuccess)                                                                     \
            return fail((h), TQR_ERR_NCCL, "%s:%d %s -> %s", __FILE__, __LINE__, #call,            \
                        (h)->nccl->GetErrorString(r_));                                            \
    } while (0)

bool supported_nb_ib(int nb, int ib) {
    return (nb == 64 || nb == 128 || nb == 256 || nb == 512) && (ib == 16 || ib == 32) && ib <= nb;
}

// Slice width of the bulk update kernel and of the (latency-critical) lookahead column.
int w_bulk(const tqr_plan_s*) { return 32; }
int w_look(const tqr_plan_s* h) {
    if (h->w_look > 0) return h->w_look;
    return h->nb >= 256 ? 8 : 16;
}

double flops_update(const tqr_plan_s* h, int k, int ncols) {
    const double nb3 = (double)h->nb * h->nb * h->nb;
    return (double)ncols * (2.0 * nb3 + 4.0 * nb3 * (double)(h->p - k - 1));
}
double flops_panel(const tqr_plan_s* h, int k) {
    const double nb3 = (double)h->nb * h->nb * h->nb;
    return 4.0 / 3.0 * nb3 + 2.0 * nb3 * (double)(h->p - k - 1);
}

void free_owner(Owner& o) {
    cudaSetDevice(o.dev);
    auto F = [](void* p) { if (p) cudaFree(p); };
    F(o.cols_dev); F(o.tiles); F(o.Vimg); F(o.T); F(o.Vexp); F(o.flags); F(o.mflags); F(o.io);
    F(o.sc_col); F(o.sc_T); F(o.sc_Vimg); F(o.sc_Vexp); F(o.Mimg); F(o.MT); F(o.Mt);
    for (int s = 0; s < 2; ++s) { F(o.rb_M[s]); F(o.rb_MT[s]); }
    for (int s = 0; s < 2; ++s) { F(o.rb_tiles[s]); F(o.rb_T[s]); F(o.rb_V[s]); }
    F(o.cflg);
    for (auto* v : {&o.ev_panel, &o.ev_recv, &o.ev_look, &o.tp0, &o.tp1, &o.tref, &o.ev_load, &o.ev_chunk, &o.ev_dom,
                    &o.tb0, &o.tb1, &o.ev_prepanel})
        for (auto e : *v) if (e) cudaEventDestroy(e);
    for (auto e : o.tl) if (e) cudaEventDestroy(e);
    for (auto* vv : {&o.ev_u, &o.tm0, &o.tm1})
        for (auto& v : *vv) for (auto e : v) if (e) cudaEventDestroy(e);
    for (auto s : o.s_u) if (s) cudaStreamDestroy(s);
    if (o.s_panel) cudaStreamDestroy(o.s_panel);
    if (o.s_upd) cudaStreamDestroy(o.s_upd);
    if (o.s_comm) cudaStreamDestroy(o.s_comm);
    if (o.s_io) cudaStreamDestroy(o.s_io);
    if (o.s_look) cudaStreamDestroy(o.s_look);
}

// Host-side DAG (Fig. 3) per rank, the same order the executor issues.
// rank < 0: every owner is local (in-process plan) -> all owners' records.
void build_schedule(int64_t q, const std::vector<int32_t>& owner_of, int rank, std::vector<int32_t>& out) {
    for (int k = 0; k < q; ++k) {
        const int o = owner_of[k];
        if (rank < 0 || o == rank) { out.insert(out.end(), {0, k, k, k, o}); }
        out.insert(out.end(), {1, k, k, k, o});
        for (int j = k + 1; j < q; ++j)
            if (rank < 0 || owner_of[j] == rank) out.insert(out.end(), {2, k, k, j, o});
    }
}

constexpr int64_t kMaxGuide = 1 << 20;   // longest distribution guide array accepted

// Returns an empty vector when the guide would exceed kMaxGuide entries.
std::vector<int32_t> generate_guide(const std::vector<int32_t>& rates) {
    // GET_RATIO: divide by the gcd; GENERATE_ARRAY: argmax + decrement,
    // lowest ID on ties (readings Q11/Q12).
    int g = 0;
    for (int r : rates) g = std::gcd(g, r);
    std::vector<int32_t> ratio(rates.size());
    int64_t sum = 0;   // 64-bit: sum of up to ndev ratios of up to 2^31
    for (size_t i = 0; i < rates.size(); ++i) { ratio[i] = rates[i] / g; sum += ratio[i]; }
    if (sum > kMaxGuide) return {};
    std::vector<int32_t> ga(sum);
    for (int i = 0; i < sum; ++i) {
        int best = 0;
        for (int d = 1; d < (int)ratio.size(); ++d) if (ratio[d] > ratio[best]) best = d;
        ga[i] = best;
        ratio[best] -= 1;
    }
    return ga;
}

enum class Mem { Host, Device };
struct PtrInfo { Mem kind; int dev; };

PtrInfo classify(const void* p) {
    cudaPointerAttributes at;
    cudaError_t e = cudaPointerGetAttributes(&at, p);
    if (e != cudaSuccess) { cudaGetLastError(); return {Mem::Host, -1}; }
    if (at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged) return {Mem::Device, at.device};
    return {Mem::Host, -1};
}

// Entry barrier of every call that reads or writes a caller buffer: the caller may have produced
// A / B with work still queued on any stream of the device (e.g. PyTorch's current stream), and
// the plan's streams are non-blocking, so wait for the whole device first.
tqr_status sync_entry(tqr_plan h, const PtrInfo& pi) {
    int prev = -1;
    for (auto& o : h->owners) {
        if (o.dev == prev) continue;
        prev = o.dev;
        CUDA_TRY(h, cudaSetDevice(o.dev));
        CUDA_TRY(h, cudaDeviceSynchronize());
    }
    if (pi.kind == Mem::Device && pi.dev >= 0 && pi.dev != prev) {
        CUDA_TRY(h, cudaSetDevice(pi.dev));
        CUDA_TRY(h, cudaDeviceSynchronize());
    }
    return TQR_OK;
}

tqr_status ensure_io(tqr_plan h, Owner& o) {
    if (o.io || o.cols.empty()) return TQR_OK;
    CUDA_TRY(h, cudaSetDevice(o.dev));
    CUDA_TRY(h, cudaMalloc(&o.io, (size_t)h->es * h->m * h->nb * o.cols.size()));
    return TQR_OK;
}

// valid (unpadded) columns of column group j
int64_t group_cols(const tqr_plan_s* h, int64_t j) { return std::min<int64_t>(h->nb, h->n - j * h->nb); }

// Wait for a stream.  Multi-process plans poll instead of blocking, so a peer that died (its flags
// never raised, its NCCL kernels never matched) turns into an error after TQR_PEER_TIMEOUT_S
// seconds (default 600) instead of a hang; NCCL's asynchronous error is checked while polling and
// the communicator aborted on failure.  The plan is poisoned either way.
tqr_status wait_stream(tqr_plan h, cudaStream_t st) {
    if (!h->multiproc()) {
        CUDA_TRY(h, cudaStreamSynchronize(st));
        return TQR_OK;
    }
    static const double limit = [] {
        const char* e = getenv("TQR_PEER_TIMEOUT_S");
        return e ? atof(e) : 600.0;
    }();
    const auto t0 = std::chrono::steady_clock::now();
    for (int it = 0;; ++it) {
        const cudaError_t q = cudaStreamQuery(st);
        if (q == cudaSuccess) return TQR_OK;
        if (q != cudaErrorNotReady)
            return fail(h, TQR_ERR_CUDA, "stream wait: %s", cudaGetErrorString(q));
        if (h->nccl_mode && h->comm && h->nccl && h->nccl->CommGetAsyncError) {
            ncclResult_t ar = ncclSuccess;
            if (h->nccl->CommGetAsyncError(h->comm, &ar) == ncclSuccess && ar != ncclSuccess && ar != ncclInProgress) {
                if (h->nccl->CommAbort) h->nccl->CommAbort(h->comm);
                h->comm = nullptr;
                return fail(h, TQR_ERR_NCCL, "NCCL asynchronous error: %s", h->nccl->GetErrorString(ar));
            }
        }
        const double el = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
        if (el > limit) {
            if (h->nccl_mode && h->comm && h->nccl && h->nccl->CommAbort) {
                h->nccl->CommAbort(h->comm);
                h->comm = nullptr;
            }
            return fail(h, h->nccl_mode ? TQR_ERR_NCCL : TQR_ERR_CUDA,
                        "no progress from a peer rank for %.0f s (TQR_PEER_TIMEOUT_S)", el);
        }
        std::this_thread::sleep_for(std::chrono::microseconds(it < 1000 ? 20 : 200));
    }
}

tqr_status sync_all(tqr_plan h) {
    for (auto& o : h->owners) {
        CUDA_TRY(h, cudaSetDevice(o.dev));
        std::vector<cudaStream_t> ss = {o.s_panel, o.s_upd, o.s_comm, o.s_io, o.s_look};
        ss.insert(ss.end(), o.s_u.begin(), o.s_u.end());
        for (auto st : ss) {
            if (!st) continue;
            tqr_status r = wait_stream(h, st);
            if (r) return r;
        }
    }
    return TQR_OK;
}

}  // namespace

// ================================================================================= ABI
extern "C" {

const char* tqr_status_string(tqr_status s) {
    switch (s) {
        case TQR_OK: return "TQR_OK";
        case TQR_ERR_ARG: return "TQR_ERR_ARG: invalid argument";
        case TQR_ERR_ALLOC: return "TQR_ERR_ALLOC: allocation failed";
        case TQR_ERR_CUDA: return "TQR_ERR_CUDA: CUDA error";
        case TQR_ERR_NCCL: return "TQR_ERR_NCCL: NCCL error";
        case TQR_ERR_STATE: return "TQR_ERR_STATE: invalid state";
        case TQR_ERR_SINGULAR: return "TQR_ERR_SINGULAR: R has a zero diagonal entry";
        case TQR_ERR_UNSUPPORTED: return "TQR_ERR_UNSUPPORTED: not supported by this build";
    }
    return "unknown tqr_status";
}

const char* tqr_last_error(tqr_plan h) { return h ? h->err.c_str() : g_create_error.c_str(); }

static tqr_status tqr_generate_guide_impl(const int32_t* rates, int32_t ndev, int32_t* guide, int32_t cap, int32_t* len) {
    if (!rates || ndev < 1 || !len) return fail(nullptr, TQR_ERR_ARG, "generate_guide: bad arguments");
    std::vector<int32_t> r(rates, rates + ndev);
    for (int x : r) if (x <= 0) return fail(nullptr, TQR_ERR_ARG, "generate_guide: rates must be > 0");
    auto ga = generate_guide(r);
    if (ga.empty()) return fail(nullptr, TQR_ERR_ARG, "generate_guide: guide longer than %lld entries", (long long)kMaxGuide);
    *len = (int32_t)ga.size();
    if (guide) {
        if (cap < (int32_t)ga.size()) return fail(nullptr, TQR_ERR_ARG, "generate_guide: capacity %d < %zu", cap, ga.size());
        std::copy(ga.begin(), ga.end(), guide);
    }
    return TQR_OK;
}

static tqr_status validate_guide(int32_t ndev, const int32_t* guide, int32_t guide_len, std::vector<int32_t>& g) {
    if (!guide) {
        g.resize(ndev);
        for (int d = 0; d < ndev; ++d) g[d] = d;
        return TQR_OK;
    }
    if (guide_len < 1) return fail(nullptr, TQR_ERR_ARG, "guide_len must be >= 1");
    g.assign(guide, guide + guide_len);
    for (int v : g) if (v < 0 || v >= ndev) return fail(nullptr, TQR_ERR_ARG, "guide entry %d outside [0, %d)", v, ndev);
    return TQR_OK;
}

static tqr_status tqr_schedule_impl(int64_t m, int64_t n, int32_t nb, int32_t ndev, const int32_t* guide, int32_t guide_len,
                        int32_t rank, int32_t* ops, int64_t cap, int64_t* count) {
    if (m < 1 || n < 1 || m < n || nb < 1 || ndev < 1 || rank < 0 || rank >= ndev || !count)
        return fail(nullptr, TQR_ERR_ARG, "schedule: bad arguments");
    std::vector<int32_t> g;
    tqr_status st = validate_guide(ndev, guide, guide_len, g);
    if (st) return st;
    const int64_t q = (n + nb - 1) / nb;
    std::vector<int32_t> owner_of(q);
    for (int64_t j = 0; j < q; ++j) owner_of[j] = g[j % g.size()];
    std::vector<int32_t> out;
    build_schedule(q, owner_of, rank, out);
    *count = (int64_t)out.size() / 5;
    if (ops) {
        if (cap < *count) return fail(nullptr, TQR_ERR_ARG, "schedule: capacity %lld < %lld", (long long)cap, (long long)*count);
        std::copy(out.begin(), out.end(), ops);
    }
    return TQR_OK;
}

tqr_status tqr_nccl_unique_id(void* id128) {
    if (!id128) return fail(nullptr, TQR_ERR_ARG, "nccl_unique_id: NULL");
    const char* why = nullptr;
    const tqr::NcclApi* api = tqr::nccl_api(&why);
    if (!api) return fail(nullptr, TQR_ERR_NCCL, "NCCL unavailable: %s", why);
    ncclUniqueId id;
    if (api->GetUniqueId(&id) != ncclSuccess) return fail(nullptr, TQR_ERR_NCCL, "ncclGetUniqueId failed");
    std::memcpy(id128, &id, sizeof(id));
    return TQR_OK;
}

tqr_status tqr_create(int64_t m, int64_t n, int32_t nb, int32_t ib, tqr_dtype dtype, int32_t ndev,
                      const int32_t* guide, int32_t guide_len, tqr_plan* out) {
    return tqr_create_ex(m, n, nb, ib, dtype, ndev, guide, guide_len, nullptr, out);
}

static void ipc_release(tqr_plan h) {
    for (void* p : h->ipc_opened) cudaIpcCloseMemHandle(p);
    h->ipc_opened.clear();
    h->peers.clear();
    if (h->flags64) cudaFree(h->flags64);
    h->flags64 = nullptr;
    if (h->rep) { tqr_destroy(h->rep); h->rep = nullptr; }
    cudaGetLastError();
}

tqr_status tqr_destroy(tqr_plan h) {
    if (!h) return TQR_OK;
    if (h->rs) {
        if (h->rs_stream) cudaStreamSynchronize(h->rs_stream);
        ipc_release(h);
        for (size_t i = 0; i < h->kids.size(); ++i) {
            cudaSetDevice(h->kid_dev[i]);
            tqr_destroy(h->kids[i]);
            if (h->rs_zero[i]) cudaFree(h->rs_zero[i]);
        }
        if (h->top) { cudaSetDevice(h->top_dev); tqr_destroy(h->top); }
        if (h->stk) cudaFree(h->stk);
        if (h->rs_send) cudaFree(h->rs_send);
        if (h->rs_recv) cudaFree(h->rs_recv);
        if (h->rs_stream) cudaStreamDestroy(h->rs_stream);
        if (h->comm && h->nccl) h->nccl->CommDestroy(h->comm);
        cudaGetLastError();
        delete h;
        return TQR_OK;
    }
    for (auto& o : h->owners) {
        cudaSetDevice(o.dev);
        if (o.s_panel) cudaStreamSynchronize(o.s_panel);
        if (o.s_upd) cudaStreamSynchronize(o.s_upd);
        if (o.s_comm) cudaStreamSynchronize(o.s_comm);
        for (auto su : o.s_u) cudaStreamSynchronize(su);
    }
    if (h->comm && h->nccl) h->nccl->CommDestroy(h->comm);
    if (!h->owners.empty()) cudaSetDevice(h->owners[0].dev);
    ipc_release(h);
    if (h->bw) cudaFree(h->bw);
    if (h->dflag) cudaFree(h->dflag);
    if (h->prog) cudaFree(h->prog);
    for (auto& o : h->owners) free_owner(o);
    cudaGetLastError();
    delete h;
    return TQR_OK;
}

tqr_status tqr_row_split_ranges(int64_t m, int32_t nb, int32_t ndev, int64_t* r0, int64_t* rows) {
    if (m < 1 || nb < 1 || ndev < 1 || !r0 || !rows) return TQR_ERR_ARG;
    const int64_t p = (m + nb - 1) / nb;
    for (int g = 0; g < ndev; ++g) {
        const int64_t t0 = g * p / ndev, t1 = (g + 1) * p / ndev;
        r0[g] = std::min<int64_t>(t0 * nb, m);
        rows[g] = std::min<int64_t>(t1 * nb, m) - r0[g];
    }
    return TQR_OK;
}

// Row-split plan (see tqr_options.row_split): owner g holds tile rows [g p / G, (g+1) p / G).
static tqr_status create_row_split(int64_t m, int64_t n, int32_t nb, int32_t ib, tqr_dtype dtype, int32_t ndev,
                                   const tqr_options& o, bool mp, bool use_ipc, int world, tqr_plan* out) {
    const bool use_nccl = mp && !use_ipc;
    const int64_t p = (m + nb - 1) / nb;
    if (n > nb) return fail(nullptr, TQR_ERR_UNSUPPORTED, "row split: a single column tile (n <= nb) only");
    tqr_plan h = new tqr_plan_s();
    h->rs = true;
    h->m = m; h->n = n; h->nb = nb; h->ib = ib; h->p = (int)p; h->q = 1;
    h->dtype = dtype; h->ndev = ndev; h->es = (dtype == TQR_F32) ? 4 : 8;
    h->guide.assign(1, 0);
    h->owner_of.assign(1, 0);
    h->rank = mp ? o.rank : 0;
    h->world = world;
    h->nccl_mode = use_nccl;
    h->ipc_mode = use_ipc;
    h->profile = o.profile != 0;
    auto bail = [&](tqr_status st) { std::string e = h->err; tqr_destroy(h); g_create_error = e; return st; };
    h->rs_r0.resize(ndev);
    h->rs_rows.resize(ndev);
    tqr_row_split_ranges(m, nb, ndev, h->rs_r0.data(), h->rs_rows.data());
    for (int g = 0; g < ndev; ++g)
        if (h->rs_rows[g] < n) return bail(fail(h, TQR_ERR_UNSUPPORTED, "row split: owner %d gets %lld < n rows", g, (long long)h->rs_rows[g]));
    int cur = 0;
    cudaGetDevice(&cur);
    tqr_options co{};
    co.logical_devices = 1;   // each kid lives on the current device when created
    co.no_lookahead = o.no_lookahead;
    co.profile = o.profile;
    co.tree_domain = o.tree_domain;
    co.tree_group = o.tree_group;
    co.row_split = -1;
    for (int g = 0; g < ndev; ++g) {
        if (mp && g != h->rank) continue;
        const int dev = (mp || o.logical_devices) ? cur : g;
        if (cudaSetDevice(dev) != cudaSuccess) return bail(fail(h, TQR_ERR_CUDA, "cudaSetDevice(%d)", dev));
        tqr_plan kid = nullptr;
        tqr_status st = tqr_create_ex(h->rs_rows[g], n, nb, ib, dtype, 1, nullptr, 0, &co, &kid);
        if (st) return bail(fail(h, st, "row split: owner %d plan: %s", g, g_create_error.c_str()));
        h->kids.push_back(kid);
        h->kid_owner.push_back(g);
        h->kid_dev.push_back(dev);
        void* z = nullptr;
        if (cudaMalloc(&z, (size_t)h->es * n * n) != cudaSuccess || cudaMemset(z, 0, (size_t)h->es * n * n) != cudaSuccess)
            return bail(fail(h, TQR_ERR_ALLOC, "row split: zero buffer"));
        h->rs_zero.push_back(z);
        if (g == 0) {
            h->top_dev = dev;
            tqr_options to = co;
            to.tree_domain = -1;
            st = tqr_create_ex((int64_t)ndev * nb, n, nb, ib, dtype, 1, nullptr, 0, &to, &h->top);
            if (st) return bail(fail(h, st, "row split: stage-2 plan: %s", g_create_error.c_str()));
            if (cudaMalloc(&h->stk, (size_t)h->es * ndev * nb * n) != cudaSuccess)
                return bail(fail(h, TQR_ERR_ALLOC, "row split: stacked R buffer"));
        }
        if (mp) {
            if (cudaMalloc(&h->rs_send, (size_t)h->es * nb * n) != cudaSuccess ||
                (use_nccl && cudaMalloc(&h->rs_recv, (size_t)h->es * ndev * nb * n) != cudaSuccess))
                return bail(fail(h, TQR_ERR_ALLOC, "row split: gather buffers"));
        }
    }
    if (use_ipc) {
        if (cudaMalloc(&h->flags64, kFlagWords * sizeof(uint64_t)) != cudaSuccess ||
            cudaMemset(h->flags64, 0, kFlagWords * sizeof(uint64_t)) != cudaSuccess)
            return bail(fail(h, TQR_ERR_ALLOC, "IPC flag block"));
    }
    cudaSetDevice(mp || o.logical_devices ? cur : 0);
    if (cudaStreamCreateWithFlags(&h->rs_stream, cudaStreamNonBlocking) != cudaSuccess)
        return bail(fail(h, TQR_ERR_CUDA, "row split: stream"));
    if (use_nccl) {
        const char* why = nullptr;
        h->nccl = tqr::nccl_api(&why);
        if (!h->nccl) return bail(fail(h, TQR_ERR_NCCL, "NCCL unavailable: %s", why));
        ncclUniqueId id;
        std::memcpy(&id, o.nccl_id, sizeof(id));
        ncclResult_t r = h->nccl->CommInitRank(&h->comm, world, id, h->rank);
        if (r != ncclSuccess) return bail(fail(h, TQR_ERR_NCCL, "ncclCommInitRank: %s", h->nccl->GetErrorString(r)));
    }
    cudaSetDevice(cur);
    *out = h;
    return TQR_OK;
}

static tqr_status tqr_create_ex_impl(int64_t m, int64_t n, int32_t nb, int32_t ib, tqr_dtype dtype, int32_t ndev,
                         const int32_t* guide, int32_t guide_len, const tqr_options* opt, tqr_plan* out) {
    if (!out) return fail(nullptr, TQR_ERR_ARG, "out is NULL");
    *out = nullptr;
    if (m < 1 || n < 1 || m < n) return fail(nullptr, TQR_ERR_ARG, "need m >= n >= 1 (m=%lld n=%lld)", (long long)m, (long long)n);
    if (nb < 1 || ib < 1 || ib > nb || nb % ib) return fail(nullptr, TQR_ERR_ARG, "need 1 <= ib <= nb, nb %% ib == 0");
    if (dtype != TQR_F64 && dtype != TQR_F32) return fail(nullptr, TQR_ERR_ARG, "unknown dtype");
    if (ndev < 1) return fail(nullptr, TQR_ERR_ARG, "ndev must be >= 1");
    std::vector<int32_t> g;
    tqr_status st = validate_guide(ndev, guide, guide_len, g);
    if (st) return st;
    if (!supported_nb_ib(nb, ib)) return fail(nullptr, TQR_ERR_UNSUPPORTED, "nb in {64,128,256,512}, ib in {16,32} only");
    tqr_options o{};
    if (opt) o = *opt;
    // NCCL mode: world > 1, or a single-rank communicator when an nccl_id is given explicitly
    // Multi-process: world > 1, a 1-rank NCCL communicator (nccl_id), or an explicit IPC transport.
    if (o.transport < TQR_TRANSPORT_AUTO || o.transport > TQR_TRANSPORT_IPC)
        return fail(nullptr, TQR_ERR_ARG, "unknown transport %d", o.transport);
    const bool mp = o.world > 1 || o.nccl_id != nullptr || o.transport == TQR_TRANSPORT_IPC;
    const bool use_ipc = mp && (o.transport == TQR_TRANSPORT_IPC || (o.transport == TQR_TRANSPORT_AUTO && !o.nccl_id));
    const bool use_nccl = mp && !use_ipc;
    const int world = o.world > 1 ? o.world : 1;
    if (mp && (o.rank < 0 || o.rank >= world || ndev != world))
        return fail(nullptr, TQR_ERR_ARG, "multi-process: need 0 <= rank < world == ndev");
    if (use_nccl && !o.nccl_id) return fail(nullptr, TQR_ERR_ARG, "NCCL transport: nccl_id is required");
    if (use_ipc && world > kIpcMaxWorld) return fail(nullptr, TQR_ERR_ARG, "IPC transport: world > %d", kIpcMaxWorld);
    int ndevices = 0;
    if (cudaGetDeviceCount(&ndevices) != cudaSuccess || ndevices < 1) {
        cudaGetLastError();
        return fail(nullptr, TQR_ERR_CUDA, "no CUDA device");
    }
    if (!mp && !o.logical_devices && ndev > ndevices)
        return fail(nullptr, TQR_ERR_ARG, "ndev %d > %d visible CUDA devices (set logical_devices)", ndev, ndevices);

    {
        const int64_t pp = (m + nb - 1) / nb, qq = (n + nb - 1) / nb;
        const bool rs = o.row_split > 0 ||
                        (o.row_split == 0 && qq == 1 && ndev > 1 && dtype == TQR_F64 && pp >= 2 * ndev);
        if (rs) return create_row_split(m, n, nb, ib, dtype, ndev, o, mp, use_ipc, world, out);
    }
    tqr_plan h = new tqr_plan_s();
    h->m = m; h->n = n; h->nb = nb; h->ib = ib; h->p = (int)((m + nb - 1) / nb); h->q = (int)((n + nb - 1) / nb);
    h->dtype = dtype; h->ndev = ndev; h->guide = g;
    h->es = (dtype == TQR_F32) ? 4 : 8;
    h->vt = (dtype == TQR_F32) ? tqr::f32_img_tile(nb, ib) : (int64_t)nb * nb;
    h->logical = o.logical_devices != 0;
    h->rank = mp ? o.rank : 0;
    h->world = world;
    h->nccl_mode = use_nccl;
    h->ipc_mode = use_ipc;
    h->lookahead = o.no_lookahead == 0;
    h->profile = o.profile != 0;
    if (const char* e = getenv("TQR_LA_OVERLAP")) h->la_overlap = atoi(e) != 0;
    if (const char* e = getenv("TQR_W16")) h->w16 = atoi(e) != 0;
    if (const char* e = getenv("TQR_CRITICAL_PATH_PROBE")) h->cp_probe = atoi(e) != 0;
    if (const char* e = getenv("TQR_W_LOOK")) { int v = atoi(e); if (v == 8 || v == 16 || v == 32) h->w_look = v; }
    if (const char* e = getenv("TQR_UPDATE_STREAMS")) { int v = atoi(e); if (v >= 1 && v <= 16) h->nstreams = v; }
    // Tree mode (NEXT-1): TS domains of L tiles factored one per CTA, merged by a flat TT chain.
    // Auto: a single panel column (q == 1, e.g. C4) whose flat chain has parallelism 1.
    if (o.tree_domain > 0) h->tree_L = o.tree_domain;
    else if (o.tree_domain == 0 && h->q == 1 && h->p >= 8) {
        int sms = 148;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
        h->tree_L = std::max(2, (h->p + sms - 1) / sms);
    }
    if (h->tree_L >= h->p) h->tree_L = 0;
    // Domain phase: a single CTA per domain pays ~2 ms per nb = 512 tile but runs one domain per
    // SM -- right for many long domains (C4); a few short domains run faster as wavefront jobs.
    if (h->tree_L > 0) {
        int sms = 148;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
        h->tree_one_cta = h->ndom(0) * 2 > sms;
        if (const char* e = getenv("TQR_TREE_ONE_CTA")) h->tree_one_cta = atoi(e) != 0;
        const int nblk = nb / ib;
        const int D0 = h->ndom(0);
        h->tree_split = (D0 * nblk * 5 <= sms) ? 4 : (D0 * nblk * 3 <= sms ? 2 : 1);
        if (ib < 32 && h->tree_split > 2) h->tree_split = 2;
        if (ib / h->tree_split < 8) h->tree_split = 1;
        if (const char* e = getenv("TQR_TREE_SPLIT")) { int v = atoi(e); if (v == 1 || v == 2 || v == 4) h->tree_split = v; }
    }
    if (h->tree_L > 0 && dtype != TQR_F64) { h->tree_L = 0; if (o.tree_domain > 0) { delete h; return fail(nullptr, TQR_ERR_UNSUPPORTED, "tree mode: FP64 only in this build"); } }
    h->dmax = h->ndom(0);
    // Merge tree of the D domain heads: per level, groups of G heads merged concurrently (D - 1
    // sequential merges -> (G - 1) * ceil(log_G D)); default G ~ sqrt(D) (two levels).
    if (h->tree_L > 0) {
        const int D0 = h->dmax;
        if (o.tree_group > 1) h->tree_G = o.tree_group;
        else if (o.tree_group == 0 && D0 >= 16) h->tree_G = (int)std::ceil(std::sqrt((double)D0));
        if (const char* e = getenv("TQR_TREE_GROUP")) h->tree_G = atoi(e);
        if (h->tree_G < 2) h->tree_G = 0;
        h->merge_split = (ib >= 32) ? 2 : 1;
        if (const char* e = getenv("TQR_MERGE_SPLIT")) { int v = atoi(e); if (v == 1 || v == 2 || v == 4) h->merge_split = v; }
        if (ib / h->merge_split < 8) h->merge_split = 1;
    }
    // Panel sub-slicing: split the apply chain of each ib column block over 4 CTAs when the
    // panel is on the critical path (few trailing columns per panel step or several owners).
    // measured (r02): 4 sub-slices (W = 8) cut the C5 8-owner critical path 417 -> 345 ms and C3
    // 236.9 -> 232.1 ms (the last column blocks' sequential applies bound the TS wavefront); a single
    // owner with many columns (C5 on one GPU: panels hidden behind the updates) keeps 2 (1640 vs 1646 ms:
    // fewer SMs taken from the bulk update)
    h->panel_split = (ndev == 1 && h->q > 32) ? 2 : 4;
    if (ib < 32 && h->panel_split > 2) h->panel_split = 2;
    if (const char* e = getenv("TQR_PANEL_SPLIT")) { int v = atoi(e); if (v == 1 || v == 2 || v == 4) h->panel_split = v; }
    if (ib / h->panel_split < 8) h->panel_split = 1;
    {
        // The overlapped lookahead's CTAs spin until the panel publishes tiles; forward progress needs
        // the whole panel grid resident beside them (one CTA per SM each; fewer SMs under MPS / a
        // partitioned GPU): otherwise the lookahead waits for the panel on the stream instead.
        int sms = 148;
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
        const int panel_ctas = (nb / ib) * (h->panel_split + 1);
        const int look_ctas = nb / w_look(h);
        h->la_fits = panel_ctas + look_ctas <= sms;
    }
    {
        // Remote trailing lookahead: the owner of column k+1 (another owner) receives panel k in chunks
        // of tiles as the TS chain publishes them and starts its lookahead on the first chunk.  Logical
        // owners and IPC ranks on distinct GPUs by default (IPC ranks sharing a GPU: off, decided in
        // tqr_ipc_connect); in-process owners on several GPUs and NCCL: opt-in / off.
        const char* e = getenv("TQR_LA_REMOTE");
        const int want = e ? atoi(e) : -1;
        const bool path = h->logical || use_ipc || (want > 0 && !use_nccl);
        h->la_remote = want != 0 && path && h->lookahead && dtype == TQR_F64 && h->tree_L == 0 && ndev > 1 &&
                       h->la_fits;
        h->la_chunk = std::max(8, (h->p + kMaxChunks - 1) / kMaxChunks);
    }
    h->owner_of.resize(h->q);
    for (int j = 0; j < h->q; ++j) h->owner_of[j] = g[j % g.size()];

    int cur = 0;
    cudaGetDevice(&cur);
    const int nown = mp ? 1 : ndev;
    h->owners.resize(nown);
    auto bail = [&](tqr_status s) { std::string e = h->err; tqr_destroy(h); g_create_error = e; return s; };
    int prio_lo = 0, prio_hi = 0;
    cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi);
    const int64_t p = h->p, tile = (int64_t)nb * nb, tsz = (int64_t)ib * nb;
    for (int li = 0; li < nown; ++li) {
        Owner& ow = h->owners[li];
        ow.id = mp ? h->rank : li;
        ow.dev = (mp || h->logical) ? cur : li;
        ow.lidx.assign(h->q, -1);
        for (int j = 0; j < h->q; ++j)
            if (h->owner_of[j] == ow.id) { ow.lidx[j] = (int32_t)ow.cols.size(); ow.cols.push_back(j); }
        if (cudaSetDevice(ow.dev) != cudaSuccess) return bail(fail(h, TQR_ERR_CUDA, "cudaSetDevice(%d)", ow.dev));
        auto mk = [&](cudaStream_t* s, int prio) { return cudaStreamCreateWithPriority(s, cudaStreamNonBlocking, prio); };
        // the overlapped lookahead (it spins on the panel's flags) one priority level below the panel,
        // so freed SMs go to the panel's CTAs first (prio_hi is the numerically smallest value)
        const int prio_look = std::min(prio_lo, prio_hi + 1);
        if (mk(&ow.s_panel, prio_hi) || mk(&ow.s_upd, prio_lo) || mk(&ow.s_comm, prio_hi) || mk(&ow.s_io, prio_hi) ||
            mk(&ow.s_look, prio_look))
            return bail(fail(h, TQR_ERR_CUDA, "stream creation failed"));
        const int S = h->nstreams_alloc();
        ow.s_u.assign(S, nullptr);
        for (auto& su : ow.s_u)
            if (mk(&su, prio_lo)) return bail(fail(h, TQR_ERR_CUDA, "stream creation failed"));
        auto mkev = [&](std::vector<cudaEvent_t>& v, int cnt, bool timing) -> bool {
            v.assign(cnt, nullptr);
            for (auto& e : v)
                if ((timing ? cudaEventCreate(&e) : cudaEventCreateWithFlags(&e, cudaEventDisableTiming)) != cudaSuccess)
                    return false;
            return true;
        };
        bool ok = mkev(ow.ev_panel, h->q, false) && mkev(ow.ev_recv, h->q, false) && mkev(ow.ev_look, h->q, false) &&
                  mkev(ow.ev_load, (int)ow.cols.size(), false) && mkev(ow.ev_prepanel, h->q, false);
        ow.ev_u.resize(S);
        for (int u = 0; u < S && ok; ++u) ok = mkev(ow.ev_u[u], h->q, false);
        if (ok && h->profile) {
            ow.tm0.resize(S); ow.tm1.resize(S); ow.tm_used.assign(S, std::vector<char>(h->q, 0));
            for (int u = 0; u < S && ok; ++u) ok = mkev(ow.tm0[u], h->q, true) && mkev(ow.tm1[u], h->q, true);
            ok = ok && mkev(ow.tp0, h->q, true) && mkev(ow.tp1, h->q, true) && mkev(ow.tref, 1, true) &&
                 mkev(ow.tb0, h->q, true) && mkev(ow.tb1, h->q, true);
            for (auto& e : ow.tl) ok = ok && cudaEventCreate(&e) == cudaSuccess;
            ow.tp_used.assign(h->q, 0);
            ow.tb_used.assign(h->q, 0);
        }
        if (!ok) return bail(fail(h, TQR_ERR_CUDA, "event creation failed"));
        const size_t nc = ow.cols.size();
        const int64_t vt = h->vt;
        auto allocb = [&](void** ptr, size_t bytes) -> bool {
            if (bytes == 0) return true;
            if (cudaMalloc(ptr, bytes) != cudaSuccess) { cudaGetLastError(); return false; }
            if (cudaMemset(*ptr, 0, bytes) != cudaSuccess) { cudaGetLastError(); return false; }
            return true;
        };
        auto alloc = [&](void** ptr, size_t elems) -> bool { return allocb(ptr, elems * h->es); };
        auto alloc64 = [&](double** ptr, size_t elems) -> bool { return allocb((void**)ptr, elems * sizeof(double)); };
        if (!alloc(&ow.tiles, nc * p * tile) || !alloc(&ow.Vimg, nc * p * vt) || !alloc(&ow.T, nc * p * tsz) ||
            !alloc(&ow.Vexp, nc * vt))
            return bail(fail(h, TQR_ERR_ALLOC, "tile storage allocation failed"));
        if (nc && h->tree_L > 0 &&
            (!alloc(&ow.Mimg, nc * h->dmax * vt) || !alloc(&ow.MT, nc * h->dmax * tsz) ||
             !alloc64(&ow.Mt, h->dmax * tile)))
            return bail(fail(h, TQR_ERR_ALLOC, "tree merge storage allocation failed"));
        if (nc && h->f32() &&
            (!alloc64(&ow.sc_col, p * tile) || !alloc64(&ow.sc_T, p * tsz) || !alloc64(&ow.sc_Vimg, p * tile) ||
             !alloc64(&ow.sc_Vexp, tile)))
            return bail(fail(h, TQR_ERR_ALLOC, "FP64 panel scratch allocation failed"));
        if (nc) {
            if (cudaMalloc(&ow.cols_dev, nc * sizeof(int32_t)) != cudaSuccess ||
                cudaMemcpy(ow.cols_dev, ow.cols.data(), nc * sizeof(int32_t), cudaMemcpyHostToDevice) != cudaSuccess)
                return bail(fail(h, TQR_ERR_ALLOC, "cols allocation failed"));
        }
        // receive slots are needed when some remote panel k precedes an owned column
        bool need_rb = use_nccl;    // every rank takes part in every ncclBroadcast
        for (int k = 0; k < h->q && !need_rb; ++k)
            if (h->owner_of[k] != ow.id)
                for (int j = k + 1; j < h->q; ++j) if (h->owner_of[j] == ow.id) { need_rb = true; break; }
        if (need_rb)
            for (int s = 0; s < 2; ++s)
                if (!alloc(&ow.rb_tiles[s], p * vt) || !alloc(&ow.rb_T[s], p * tsz) || !alloc(&ow.rb_V[s], vt) ||
                    (h->tree_L > 0 && (!alloc(&ow.rb_M[s], h->dmax * vt) || !alloc(&ow.rb_MT[s], h->dmax * tsz))))
                    return bail(fail(h, TQR_ERR_ALLOC, "receive buffer allocation failed"));
        if (nc) {
            const size_t nfl = (size_t)p * (nb / ib) * 5;   // F + up to 4 sub-slice flags
            if (cudaMalloc(&ow.flags, nfl * sizeof(unsigned)) != cudaSuccess ||
                cudaMemset(ow.flags, 0, nfl * sizeof(unsigned)) != cudaSuccess)
                return bail(fail(h, TQR_ERR_ALLOC, "flag allocation failed"));
            if (h->tree_L > 0 && (cudaMalloc(&ow.mflags, nfl * sizeof(unsigned)) != cudaSuccess ||
                                  cudaMemset(ow.mflags, 0, nfl * sizeof(unsigned)) != cudaSuccess))
                return bail(fail(h, TQR_ERR_ALLOC, "flag allocation failed"));
        }
        if (h->la_remote && !use_ipc) {
            if (cudaMalloc(&ow.cflg, 2 * kMaxChunks * sizeof(unsigned long long)) != cudaSuccess ||
                cudaMemset(ow.cflg, 0, 2 * kMaxChunks * sizeof(unsigned long long)) != cudaSuccess)
                return bail(fail(h, TQR_ERR_ALLOC, "chunk flag allocation failed"));
        }
    }
    // peer access between physical owners (single-process, several GPUs)
    if (use_ipc) {
        cudaSetDevice(cur);
        if (cudaMalloc(&h->flags64, kFlagWords * sizeof(uint64_t)) != cudaSuccess ||
            cudaMemset(h->flags64, 0, kFlagWords * sizeof(uint64_t)) != cudaSuccess)
            return bail(fail(h, TQR_ERR_ALLOC, "IPC flag block"));
    }
    if (!mp && !h->logical && ndev > 1) {
        for (int a = 0; a < ndev; ++a)
            for (int b = 0; b < ndev; ++b) {
                if (a == b) continue;
                int can = 0;
                cudaDeviceCanAccessPeer(&can, a, b);
                if (can) { cudaSetDevice(a); cudaDeviceEnablePeerAccess(b, 0); cudaGetLastError(); }
            }
    }
    if (use_nccl) {
        const char* why = nullptr;
        h->nccl = tqr::nccl_api(&why);
        if (!h->nccl) return bail(fail(h, TQR_ERR_NCCL, "NCCL unavailable: %s", why));
        ncclUniqueId id;
        std::memcpy(&id, o.nccl_id, sizeof(id));
        cudaSetDevice(cur);
        ncclResult_t r = h->nccl->CommInitRank(&h->comm, world, id, h->rank);
        if (r != ncclSuccess) return bail(fail(h, TQR_ERR_NCCL, "ncclCommInitRank: %s", h->nccl->GetErrorString(r)));
    }
    cudaSetDevice(cur);
    *out = h;
    return TQR_OK;
}

// ------------------------------------------------------------------ CUDA-IPC transport handshake
namespace {
int plan_device(tqr_plan h) {
    if (!h->owners.empty()) return h->owners[0].dev;
    if (!h->kid_dev.empty()) return h->kid_dev[0];
    int d = 0;
    cudaGetDevice(&d);
    return d;
}
cudaStream_t plan_comm_stream(tqr_plan h) { return h->rs ? h->rs_stream : h->owners[0].s_comm; }
// pointers a peer needs, in IpcSlot order (null = not allocated on this rank)
void export_ptrs(tqr_plan h, void* out[kNH]) {
    for (int i = 0; i < kNH; ++i) out[i] = nullptr;
    out[H_FLAGS] = h->flags64;
    if (h->rs) {
        out[H_RSSEND] = h->rs_send;
        return;
    }
    Owner& o = h->owners[0];
    for (int sl = 0; sl < 2; ++sl) {
        out[H_RB + 5 * sl + 0] = o.rb_tiles[sl];
        out[H_RB + 5 * sl + 1] = o.rb_T[sl];
        out[H_RB + 5 * sl + 2] = o.rb_V[sl];
        out[H_RB + 5 * sl + 3] = o.rb_M[sl];
        out[H_RB + 5 * sl + 4] = o.rb_MT[sl];
    }
    out[H_TILES] = o.tiles; out[H_VIMG] = o.Vimg; out[H_T] = o.T; out[H_VEXP] = o.Vexp;
    out[H_MIMG] = o.Mimg; out[H_MT] = o.MT;
}
void peer_from_ptrs(IpcPeer& pr, void* const ptr[kNH]) {
    pr.flags = static_cast<uint64_t*>(ptr[H_FLAGS]);
    for (int sl = 0; sl < 2; ++sl)
        for (int f = 0; f < 5; ++f) pr.rb[sl][f] = ptr[H_RB + 5 * sl + f];
    for (int f = 0; f < 6; ++f) pr.st[f] = ptr[H_TILES + f];
    pr.rs_send = ptr[H_RSSEND];
}
}  // namespace

static tqr_status tqr_ipc_handle_impl(tqr_plan h, void* buf, int64_t cap, int64_t* len) {
    if (!h || !len) return fail(h, TQR_ERR_ARG, "ipc_handle: bad arguments");
    if (!h->ipc_mode) return fail(h, TQR_ERR_STATE, "ipc_handle: the plan does not use the IPC transport");
    *len = (int64_t)sizeof(IpcBlob);
    if (!buf) return TQR_OK;
    if (cap < *len) return fail(h, TQR_ERR_ARG, "ipc_handle: capacity %lld < %lld", (long long)cap, (long long)*len);
    IpcBlob b;
    std::memset(&b, 0, sizeof(b));
    b.magic = kIpcMagic;
    b.rank = h->rank;
    b.world = h->world;
    b.dev = plan_device(h);
    {
        cudaDeviceProp pr;
        CUDA_TRY(h, cudaGetDeviceProperties(&pr, b.dev));
        std::memcpy(b.uuid, &pr.uuid, sizeof(b.uuid));
    }
    void* ptr[kNH];
    export_ptrs(h, ptr);
    CUDA_TRY(h, cudaSetDevice(b.dev));
    for (int i = 0; i < kNH; ++i)
        if (ptr[i]) {
            CUDA_TRY(h, cudaIpcGetMemHandle(&b.h[i], ptr[i]));
            b.present |= 1ull << i;
        }
    std::memcpy(buf, &b, sizeof(b));
    return TQR_OK;
}

static tqr_status tqr_ipc_connect_impl(tqr_plan h, const void* all, int64_t len) {
    if (!h || !all) return fail(h, TQR_ERR_ARG, "ipc_connect: bad arguments");
    if (!h->ipc_mode) return fail(h, TQR_ERR_STATE, "ipc_connect: the plan does not use the IPC transport");
    if (h->ipc_connected) return fail(h, TQR_ERR_STATE, "ipc_connect: already connected");
    const int64_t bs = (int64_t)sizeof(IpcBlob);
    if (len != bs * h->world) return fail(h, TQR_ERR_ARG, "ipc_connect: %lld bytes, expected %lld", (long long)len, (long long)(bs * h->world));
    const int dev = plan_device(h);
    CUDA_TRY(h, cudaSetDevice(dev));
    h->peers.assign(h->world, IpcPeer());
    for (int r = 0; r < h->world; ++r) {
        IpcBlob b;
        std::memcpy(&b, static_cast<const char*>(all) + r * bs, sizeof(b));
        if (b.magic != kIpcMagic || b.rank != r || b.world != h->world)
            return fail(h, TQR_ERR_ARG, "ipc_connect: blob %d is not rank %d's export", r, r);
        void* ptr[kNH];
        if (r == h->rank) {
            export_ptrs(h, ptr);
        } else {
            for (int i = 0; i < kNH; ++i) {
                ptr[i] = nullptr;
                if (b.present >> i & 1ull) {
                    CUDA_TRY(h, cudaIpcOpenMemHandle(&ptr[i], b.h[i], cudaIpcMemLazyEnablePeerAccess));
                    h->ipc_opened.push_back(ptr[i]);
                }
            }
        }
        peer_from_ptrs(h->peers[r], ptr);
        h->peers[r].dev = b.dev;
        std::memcpy(h->peers[r].uuid, b.uuid, sizeof(b.uuid));
    }
    // ranks sharing a GPU are time-sliced: a lookahead spinning on another rank's chunk flags would
    // hold its context's slice -- no remote trailing then (same decision on every rank: all devices known)
    // (TQR_LA_REMOTE=2 forces it anyway: the multi-process tests exercise the chunked IPC path on one GPU)
    const char* lr = getenv("TQR_LA_REMOTE");
    if (!(lr && atoi(lr) == 2))
        for (int a = 0; a < h->world; ++a)
            for (int b = a + 1; b < h->world; ++b)
                if (std::memcmp(h->peers[a].uuid, h->peers[b].uuid, sizeof(h->peers[a].uuid)) == 0) h->la_remote = false;
    // arm: my receive slots 0 / 1 are free for steps 0 / 1 of the first factorization, at every
    // possible root (the flag lives in the root's block; roots only ever wait on their own block)
    cudaStream_t s = plan_comm_stream(h);
    for (int d = 0; d < h->world; ++d) {
        if (d == h->rank) continue;
        for (int sl = 0; sl < 2; ++sl)
            CUDA_TRY(h, tqr::sig_write(s, h->peers[d].flags + F_FREED + 2 * h->rank + sl, (uint64_t)h->epoch + 1 + sl));
    }
    CUDA_TRY(h, cudaStreamSynchronize(s));
    h->ipc_connected = true;
    return TQR_OK;
}

tqr_status tqr_issued_ops(tqr_plan h, int32_t* ops, int64_t cap, int64_t* count) {
    if (!h || !count) return fail(h, TQR_ERR_ARG, "issued_ops: bad arguments");
    *count = (int64_t)h->issued.size() / 5;
    if (ops) {
        if (cap < *count) return fail(h, TQR_ERR_ARG, "issued_ops: capacity %lld < %lld", (long long)cap, (long long)*count);
        std::copy(h->issued.begin(), h->issued.end(), ops);
    }
    return TQR_OK;
}

int32_t tqr_plan_flags(tqr_plan h) {
    if (!h) return 0;
    int32_t f = 0;
    if (h->rs) f |= TQR_PLAN_ROW_SPLIT;
    if (h->tree_L > 0 || (h->rs && !h->kids.empty() && h->kids[0]->tree_L > 0)) f |= TQR_PLAN_TREE;
    if (h->multiproc()) f |= TQR_PLAN_MULTIPROC;
    if (h->ipc_mode) f |= TQR_PLAN_IPC;
    if (h->nccl_mode) f |= TQR_PLAN_NCCL;
    if (h->f32()) f |= TQR_PLAN_F32;
    return f;
}

int32_t tqr_owner(tqr_plan h, int64_t j) {
    if (!h || j < 0 || j >= h->q) return -1;
    return h->owner_of[j];
}

int64_t tqr_launch_count(tqr_plan h) {
    if (!h) return 0;
    int64_t c = h->launches;
    for (auto k : h->kids) c += tqr_launch_count(k);
    if (h->top) c += tqr_launch_count(h->top);
    h->launches = 0;
    return c;
}

tqr_status tqr_kernel_stats(tqr_plan h, int32_t which, int64_t* count, double* ms, double* flops, int32_t reset) {
    if (!h || which < 0 || which > 3) return fail(h, TQR_ERR_ARG, "kernel_stats: bad arguments");
    if (h->rs) {   // the owners' row blocks run concurrently: count and flops add, time is the max
        int64_t c = 0;
        double t = 0.0, f = 0.0;
        std::vector<tqr_plan> all(h->kids);
        if (h->top) all.push_back(h->top);
        for (size_t i = 0; i < all.size(); ++i) {
            int64_t ci = 0;
            double ti = 0.0, fi = 0.0;
            tqr_kernel_stats(all[i], which, &ci, &ti, &fi, reset);
            c += ci;
            f += fi;
            t = (all[i] == h->top) ? t + ti : std::max(t, ti);
        }
        if (count) *count = c;
        if (ms) *ms = t;
        if (flops) *flops = f;
        return TQR_OK;
    }
    if (count) *count = h->stats[which].count;
    if (ms) *ms = h->stats[which].ms;
    if (flops) *flops = h->stats[which].flops;
    if (reset) h->stats[which] = KStat();
    return TQR_OK;
}

// ------------------------------------------------------------------ typed launch helpers
namespace {
cudaError_t to_tiles(const tqr_plan_s* h, const void* src, int64_t lda, int64_t gstride, void* dst, const int32_t* cols,
                     int local_src, int nc, cudaStream_t s) {
    const int64_t colsz = (int64_t)h->p * h->nb * h->nb;
    if (h->f32())
        return tqr::launch_to_tiles<float>((const float*)src, lda, gstride, (float*)dst, cols, local_src, nc, colsz,
                                           h->nb, h->p, h->m, h->n, s);
    return tqr::launch_to_tiles<double>((const double*)src, lda, gstride, (double*)dst, cols, local_src, nc, colsz,
                                        h->nb, h->p, h->m, h->n, s);
}
cudaError_t from_tiles(const tqr_plan_s* h, void* dst, int64_t lda, int64_t gstride, const void* src,
                       const int32_t* cols, int nc, int64_t m_rows, int64_t n_valid, int local_dst, cudaStream_t s) {
    const int64_t colsz = (int64_t)h->p * h->nb * h->nb;
    if (h->f32())
        return tqr::launch_from_tiles<float>((float*)dst, lda, gstride, (const float*)src, cols, nc, colsz, h->nb,
                                             m_rows, n_valid, local_dst, s);
    return tqr::launch_from_tiles<double>((double*)dst, lda, gstride, (const double*)src, cols, nc, colsz, h->nb,
                                          m_rows, n_valid, local_dst, s);
}
// Reflector data of panel k as seen by an update: images V (tile i at V + i*vt), T (tile i at
// T + i*ib*nb), explicit V of the diagonal tile; tree mode: merge images / T (slot e).
struct PanelRefs {
    void* V;
    void* T;
    void* Vexp;
    void* M = nullptr;
    void* MT = nullptr;
};
// One update-kernel launch: reflector tiles k_head (UNMQR, if do_unmqr) and k_head+1..p_end-1
// (TSMQR against row tile k_head) applied to nslices column slices of X.
cudaError_t update1(const tqr_plan_s* h, const void* V, const void* T, const void* Vexp, void* X, int64_t col_stride,
                    int64_t tile_stride, int64_t ld, int group0, int gstride, int k_head, int p_end, int do_unmqr,
                    int w, int nslices, bool trans, cudaStream_t s, int vstride = 1,
                    const unsigned* wflags = nullptr, unsigned wepoch = 0, int domL = 0, int njobs = 1,
                    const unsigned long long* cflags = nullptr, unsigned long long cval = 0, int cchunk = 1) {
    if (h->f32()) {
        tqr::UpdateArgsT<float> u;
        u.V = (const float*)V; u.T = (const float*)T; u.Vexp = (const float*)Vexp; u.X = (float*)X;
        u.col_stride = col_stride; u.tile_stride = tile_stride; u.ld = ld;
        u.group0 = group0; u.gstride = gstride; u.k = k_head; u.p = p_end; u.do_unmqr = do_unmqr;
        return tqr::launch_update_f32(h->nb, h->ib, w, u, nslices, trans, s);
    }
    tqr::UpdateArgs u;
    u.V = (const double*)V; u.T = (const double*)T; u.Vexp = (const double*)Vexp; u.X = (double*)X;
    u.col_stride = col_stride; u.tile_stride = tile_stride; u.ld = ld;
    u.group0 = group0; u.gstride = gstride; u.k = k_head; u.p = p_end; u.do_unmqr = do_unmqr; u.vstride = vstride;
    u.wflags = wflags; u.wepoch = wepoch;
    u.cflags = cflags; u.cval = cval; u.cchunk = cchunk;
    u.w16 = h->w16 ? 1 : 0;
    if (domL > 0) { u.domL = domL; u.nslc = nslices; }
    return tqr::launch_update(h->nb, h->ib, w, u, nslices * njobs, trans, s);
}
// Q_k^T (trans) or Q_k applied to X.  Flat: one launch (UNMQR(k) + TSMQR(k+1..p-1)).  Tree (D > 1
// domains of L tiles): per domain d, UNMQR of its head k + d*L and TSMQR of its tiles against the
// head; then the merge chain TSMQR(head_e against head_0), e = 1..D-1 (row tiles k + e*L, i.e.
// stride L*tile_stride) -- or, with groups of G domains (two-level merge), per group g the chain
// of heads gG+1..gG+G-1 against head gG, then the chain of group heads G, 2G, .. against head 0
// (merge slot e holds the reflectors of the merge whose bottom was head e).  Q is applied in the
// reverse order.  Returns the number of launches in *nl.
cudaError_t update(const tqr_plan_s* h, const PanelRefs& r, void* X, int64_t col_stride, int64_t tile_stride,
                   int64_t ld, int group0, int gstride, int k, int w, int nslices, bool trans, cudaStream_t s,
                   int64_t* nl = nullptr, const unsigned* wflags = nullptr, unsigned wepoch = 0,
                   const unsigned long long* cflags = nullptr, unsigned long long cval = 0, int cchunk = 1) {
    const int D = h->ndom(k), L = h->tree_L;
    if (D == 1) {
        if (nl) *nl += 1;
        return update1(h, r.V, r.T, r.Vexp, X, col_stride, tile_stride, ld, group0, gstride, k, h->p, 1, w, nslices,
                       trans, s, 1, wflags, wepoch, 0, 1, cflags, cval, cchunk);
    }
    // all D domains in one launch (independent row ranges; job d = domain d, head k + d*L)
    auto doms = [&]() {
        return update1(h, r.V, r.T, r.Vexp, X, col_stride, tile_stride, ld, group0, gstride, k, h->p, 1, w, nslices,
                       trans, s, 1, nullptr, 0, L, D);
    };
    // merge level of stride S (heads 0, S, 2S, .. of the domain heads, row tiles k + i*S*L, merge
    // slots i*S): jobs of G consecutive heads, each the chain of heads gG+1.. against head gG
    const int G = h->merge_group(D);
    std::vector<int64_t> lv;
    for (int64_t S = 1; S < D; S *= G) lv.push_back(S);
    auto level = [&](int64_t S) {
        const int H = (int)((D + S - 1) / S), nj = (H + G - 1) / G;
        return update1(h, r.M, r.MT, r.M, h->at(X, (int64_t)k * tile_stride), col_stride, tile_stride * L * S, ld,
                       group0, gstride, 0, H, 0, w, nslices, trans, s, (int)S, nullptr, 0, nj > 1 ? G : 0, nj);
    };
    if (nl) *nl += 1 + (int64_t)lv.size();
    cudaError_t e = cudaSuccess;
    if (trans) {   // Q^T: domains, then the merge levels bottom-up
        e = doms();
        for (size_t l = 0; l < lv.size() && e == cudaSuccess; ++l) e = level(lv[l]);
    } else {       // Q: the merge levels top-down, then the domains
        for (size_t l = lv.size(); l-- > 0 && e == cudaSuccess;) e = level(lv[l]);
        if (e == cudaSuccess) e = doms();
    }
    return e;
}
PanelRefs own_refs(const tqr_plan_s* h, Owner& O, int lc) {
    const int64_t p = h->p, tsz = (int64_t)h->ib * h->nb;
    PanelRefs r{h->at(O.Vimg, lc * p * h->vt), h->at(O.T, lc * p * tsz), h->at(O.Vexp, lc * h->vt)};
    if (O.Mimg) {
        r.M = h->at(O.Mimg, lc * h->dmax * h->vt);
        r.MT = h->at(O.MT, lc * h->dmax * tsz);
    }
    return r;
}
PanelRefs recv_refs(const tqr_plan_s*, Owner& O, int slot) {
    return {O.rb_tiles[slot], O.rb_T[slot], O.rb_V[slot], O.rb_M[slot], O.rb_MT[slot]};
}
}  // namespace

// ------------------------------------------------------------------ row split (NEXT-1 across owners)
namespace {
tqr_status kid_fail(tqr_plan h, tqr_plan kid, tqr_status st) {
    h->poisoned = h->poisoned || st == TQR_ERR_CUDA || st == TQR_ERR_NCCL;
    return fail(h, st, "row split: %s", tqr_last_error(kid));
}
tqr_status rs_load(tqr_plan h, const void* A, int64_t lda) {
    h->factored = false;
    for (size_t i = 0; i < h->kids.size(); ++i) {
        CUDA_TRY(h, cudaSetDevice(h->kid_dev[i]));
        const int g = h->kid_owner[i];
        tqr_status st = tqr_load(h->kids[i], static_cast<const char*>(A) + h->rs_r0[g] * h->es, lda);
        if (st) return kid_fail(h, h->kids[i], st);
    }
    return TQR_OK;
}
// every owner factors its row block; the owners' R factors (tile 0 of each block) are stacked on
// owner 0 (peer copies, or an NCCL all-gather) with their reflectors zeroed, and factored again
tqr_status rs_factor(tqr_plan h) {
    if (h->ipc_mode && !h->ipc_connected) return fail(h, TQR_ERR_STATE, "IPC plan not connected (tqr_ipc_connect)");
    const int G = h->ndev, nb = h->nb;
    const int64_t n = h->n, es = h->es, ld = (int64_t)G * nb;
    for (size_t i = 0; i < h->kids.size(); ++i) {
        CUDA_TRY(h, cudaSetDevice(h->kid_dev[i]));
        tqr_status st = tqr_factor_tiles(h->kids[i]);
        if (st) return kid_fail(h, h->kids[i], st);
    }
    if (h->ipc_mode) {
        // every rank publishes its R_g (tile 0 of its block) in rs_send once rank 0 has pulled the
        // previous one; rank 0 pulls all of them into the stack (IPC reads), then releases rs_send
        const uint64_t E = ++h->rs_epoch;
        tqr_plan kid = h->kids[0];
        CUDA_TRY(h, cudaSetDevice(h->kid_dev[0]));
        cudaStream_t s = h->rs_stream;
        CUDA_TRY(h, tqr::sig_wait_geq(s, h->flags64 + F_PULLED, E - 1));
        CUDA_TRY(h, cudaMemcpyAsync(h->rs_send, kid->owners[0].tiles, (size_t)es * nb * n, cudaMemcpyDeviceToDevice, s));
        CUDA_TRY(h, tqr::sig_write(s, h->peers[0].flags + F_RSREADY + h->rank, E));
        if (h->top) {
            for (int g = 0; g < G; ++g) {
                CUDA_TRY(h, tqr::sig_wait_geq(s, h->flags64 + F_RSREADY + g, E));
                CUDA_TRY(h, cudaMemcpy2DAsync(h->at(h->stk, (int64_t)g * nb), ld * es, h->peers[g].rs_send, nb * es,
                                              nb * es, n, cudaMemcpyDefault, s));
            }
            for (int g = 0; g < G; ++g) CUDA_TRY(h, tqr::sig_write(s, h->peers[g].flags + F_PULLED, E));
        }
    } else if (h->multiproc()) {
        tqr_plan kid = h->kids[0];
        CUDA_TRY(h, cudaSetDevice(h->kid_dev[0]));
        CUDA_TRY(h, cudaMemcpyAsync(h->rs_send, kid->owners[0].tiles, (size_t)es * nb * n, cudaMemcpyDeviceToDevice,
                                    h->rs_stream));
        const ncclDataType_t dt = h->f32() ? ncclFloat32 : ncclFloat64;
        NCCL_TRY(h, h->nccl->AllGather(h->rs_send, h->rs_recv, (size_t)nb * n, dt, h->comm, h->rs_stream));
        if (h->top) {
            for (int g = 0; g < G; ++g)
                CUDA_TRY(h, cudaMemcpy2DAsync(h->at(h->stk, (int64_t)g * nb), ld * es, h->at(h->rs_recv, (int64_t)g * nb * n),
                                              nb * es, nb * es, n, cudaMemcpyDeviceToDevice, h->rs_stream));
        }
    } else {
        CUDA_TRY(h, cudaSetDevice(h->top_dev));
        for (size_t i = 0; i < h->kids.size(); ++i)
            CUDA_TRY(h, cudaMemcpy2DAsync(h->at(h->stk, (int64_t)h->kid_owner[i] * nb), ld * es,
                                          h->kids[i]->owners[0].tiles, nb * es, nb * es, n, cudaMemcpyDefault,
                                          h->rs_stream));
    }
    if (h->top) {
        CUDA_TRY(h, cudaSetDevice(h->top_dev));
        if (h->f32()) CUDA_TRY(h, tqr::launch_zero_below_blocks<float>((float*)h->stk, ld, ld, n, nb, h->rs_stream));
        else CUDA_TRY(h, tqr::launch_zero_below_blocks<double>((double*)h->stk, ld, ld, n, nb, h->rs_stream));
        h->launches++;
        { tqr_status ws = wait_stream(h, h->rs_stream); if (ws) return ws; }
        tqr_status st = tqr_load(h->top, h->stk, ld);
        if (!st) st = tqr_factor_tiles(h->top);
        if (st) return kid_fail(h, h->top, st);
    } else {
        { tqr_status ws = wait_stream(h, h->rs_stream); if (ws) return ws; }
    }
    h->factored = true;
    return TQR_OK;
}
// each owner writes its rows (R_g + zeros), then zeros over R_g; owner 0 writes the final R
tqr_status rs_store(tqr_plan h, void* A, int64_t lda) {
    const int64_t n = h->n, es = h->es, ld = (int64_t)h->ndev * h->nb;
    for (size_t i = 0; i < h->kids.size(); ++i) {
        CUDA_TRY(h, cudaSetDevice(h->kid_dev[i]));
        const int g = h->kid_owner[i];
        char* Ag = static_cast<char*>(A) + h->rs_r0[g] * es;
        tqr_status st = tqr_store_r(h->kids[i], Ag, lda);
        if (st) return kid_fail(h, h->kids[i], st);
        if (g != 0) {
            CUDA_TRY(h, cudaMemcpy2D(Ag, lda * es, h->rs_zero[i], n * es, n * es, n, cudaMemcpyDefault));
        }
    }
    if (h->top) {
        CUDA_TRY(h, cudaSetDevice(h->top_dev));
        tqr_status st = tqr_store_r(h->top, h->stk, ld);
        if (st) return kid_fail(h, h->top, st);
        CUDA_TRY(h, cudaMemcpy2D(A, lda * es, h->stk, ld * es, n * es, n, cudaMemcpyDefault));
    }
    return TQR_OK;
}
}  // namespace

// ------------------------------------------------------------------ a1: load
namespace {
// stats[2]: the layout pass just completed (ev = 0: load, 2: store) on every owner: device time of
// the slowest owner, algorithmic bytes = read + write of the owned columns (es * m * nb each way)
tqr_status layout_stat(tqr_plan h, int ev) {
    if (!h->profile) return TQR_OK;
    float mx = 0.f;
    double bytes = 0.0;
    for (auto& o : h->owners) {
        if (o.cols.empty()) continue;
        CUDA_TRY(h, cudaSetDevice(o.dev));
        float t = 0.f;
        CUDA_TRY(h, cudaEventElapsedTime(&t, o.tl[ev], o.tl[ev + 1]));
        mx = std::max(mx, t);
        bytes += 2.0 * h->es * (double)h->m * h->nb * o.cols.size();
    }
    h->stats[2].count += 1;
    h->stats[2].ms += mx;
    h->stats[2].flops += bytes;
    return TQR_OK;
}
}  // namespace

static tqr_status tqr_load_impl(tqr_plan h, const void* A, int64_t lda) {
    NvtxRange nvtx_("tqr_load (a1)");
    if (!h) return TQR_ERR_ARG;
    if (h->rs) {
        if (h->poisoned) return fail(h, TQR_ERR_STATE, "plan poisoned by an earlier CUDA/NCCL failure");
        if (!A || lda < h->m) return fail(h, TQR_ERR_ARG, "load: A is NULL or lda < m");
        return rs_load(h, A, lda);
    }
    if (h->poisoned) return fail(h, TQR_ERR_STATE, "plan poisoned by an earlier CUDA/NCCL failure");
    if (!A || lda < h->m) return fail(h, TQR_ERR_ARG, "load: A is NULL or lda < m");
    const PtrInfo pi = classify(A);
    const int64_t nb = h->nb, es = h->es;
    h->factored = false;
    { tqr_status st0 = sync_entry(h, pi); if (st0) return st0; }
    for (auto& o : h->owners) {
        if (o.cols.empty()) continue;
        CUDA_TRY(h, cudaSetDevice(o.dev));
        const int nc = (int)o.cols.size();
        if (h->profile) CUDA_TRY(h, cudaEventRecord(o.tl[0], o.s_upd));
        if (pi.kind == Mem::Device && pi.dev == o.dev) {
            CUDA_TRY(h, to_tiles(h, A, lda, nb * lda, o.tiles, o.cols_dev, 0, nc, o.s_upd));
            h->launches++;
        } else {
            tqr_status st = ensure_io(h, o);
            if (st) return st;
            for (int lc = 0; lc < nc; ++lc) {
                const int64_t j = o.cols[lc];
                CUDA_TRY(h, cudaMemcpy2DAsync(h->at(o.io, (int64_t)lc * h->m * nb), h->m * es,
                                              static_cast<const char*>(A) + j * nb * lda * es, lda * es, h->m * es,
                                              group_cols(h, j), cudaMemcpyDefault, o.s_upd));
            }
            // io holds the owned columns in local order: group lc at io + lc*m*nb
            CUDA_TRY(h, to_tiles(h, o.io, h->m, h->m * nb, o.tiles, o.cols_dev, 1, nc, o.s_upd));
            h->launches++;
        }
        if (h->profile) CUDA_TRY(h, cudaEventRecord(o.tl[1], o.s_upd));
    }
    tqr_status st = sync_all(h);
    if (st) return st;
    return layout_stat(h, 0);
}

// ------------------------------------------------------------------ a2-a7: factor
namespace {
// Union length of [t0, t1] intervals (ms) -- device-busy time of one kernel class across streams.
double union_ms(std::vector<std::pair<double, double>>& iv) {
    std::sort(iv.begin(), iv.end());
    double tot = 0.0, cs = -1e300, ce = -1e300;
    for (auto& x : iv) {
        if (x.first > ce) { if (ce > cs) tot += ce - cs; cs = x.first; ce = x.second; }
        else ce = std::max(ce, x.second);
    }
    if (ce > cs) tot += ce - cs;
    return tot;
}

// PANEL(k) on its owner's panel stream.  FP64: the panel kernel factors the owner's tiles in
// place.  FP32: widen tiles k..p-1 of the column into the FP64 scratch column, factor there,
// narrow R / reflectors / T / stage images back (qr_kernels_f32.cu).
tqr_status launch_panel_step(tqr_plan h, Owner& O, int k, unsigned epoch) {
    const int p = h->p, nb = h->nb, ib = h->ib;
    const int64_t tile = (int64_t)nb * nb, tsz = (int64_t)ib * nb, colsz = (int64_t)p * tile;
    const int lc = O.lidx[k];
    tqr::PanelArgs a;
    a.flags = O.flags;
    a.epoch = epoch;
    a.k = k;
    a.p = p;
    if (!h->f32()) {
        a.col = h->at<double>(O.tiles, lc * colsz);
        a.Vimg = h->at<double>(O.Vimg, lc * colsz);
        a.T = h->at<double>(O.T, lc * (int64_t)p * tsz);
        a.Vexp = h->at<double>(O.Vexp, lc * tile);
        const int D = h->ndom(k);
        if (D == 1) {
            CUDA_TRY(h, tqr::launch_panel(nb, ib, h->panel_split, a, O.s_panel));
            h->launches++;
            return TQR_OK;
        }
        // tree: D TS domains (one CTA each), then the flat merge chain of the domain heads' R
        // factors against head 0 (the panel kernel in TSQRT-only mode on the merge bottoms)
        if (h->domains_done) {
            // launched per row chunk by the streamed tall factor; the panel stream waited for them
        } else if (h->tree_one_cta) {
            tqr::DomainArgs da{a.col, a.T, a.Vimg, a.Vexp, k, p, h->tree_L};
            CUDA_TRY(h, tqr::launch_domains(nb, ib, da, D, O.s_panel));
        } else {
            // short domains: each domain its own wavefront (the panel kernel, one job per domain)
            tqr::PanelArgs dj = a;
            dj.L = h->tree_L;
            CUDA_TRY(h, tqr::launch_panel(nb, ib, h->tree_split, dj, O.s_panel, D));
        }
        CUDA_TRY(h, tqr::launch_merge_prep(nb, a.col, O.Mt, k, h->tree_L, D, O.s_panel));
        const PanelRefs r = own_refs(h, O, lc);
        tqr::PanelArgs m = a;
        m.col = O.Mt;
        m.T = (double*)r.MT;
        m.Vimg = (double*)r.M;
        m.Vexp = (double*)r.M;
        m.k = 0;
        m.p = D;
        m.top = a.col + (int64_t)k * tile;
        m.skip_ge = 1;
        m.flags = O.mflags;
        m.fslots = p;
        // merge tree, one launch per level of stride S: H = ceil(D/S) heads (slots 0, S, 2S, ..), jobs
        // of G consecutive heads -- job g merges heads gG+1..gG+G-1 into head gG (job 0's top is the
        // real head tile, job g > 0's is merge slot gGS); a single job is one chain (split as a panel)
        const int G = h->merge_group(D);
        int nlv = 0;
        for (int64_t S = 1; S < D; S *= G, ++nlv) {
            const int H = (int)((D + S - 1) / S), nj = (H + G - 1) / G;
            tqr::PanelArgs ml = m;
            ml.stride = (int)S;
            ml.p = H;
            ml.L = nj > 1 ? G : 0;
            CUDA_TRY(h, tqr::launch_panel(nb, ib, nj > 1 ? h->merge_split : h->panel_split, ml, O.s_panel, nj));
        }
        h->launches += 2 + nlv;
        return TQR_OK;
    }
    CUDA_TRY(h, tqr::launch_widen(h->at<float>(O.tiles, lc * colsz + k * tile), O.sc_col + k * tile,
                                  (int64_t)(p - k) * tile, O.s_panel));
    a.col = O.sc_col; a.Vimg = O.sc_Vimg; a.T = O.sc_T; a.Vexp = O.sc_Vexp;
    CUDA_TRY(h, tqr::launch_panel(nb, ib, h->panel_split, a, O.s_panel));
    const PanelRefs r = own_refs(h, O, lc);
    CUDA_TRY(h, tqr::launch_narrow_panel(nb, ib, O.sc_col, O.sc_T, h->at<float>(O.tiles, lc * colsz), (float*)r.T,
                                         (float*)r.V, (float*)r.Vexp, k, p, O.s_panel));
    h->launches += 3;
    return TQR_OK;
}
}  // namespace

static tqr_status tqr_factor_tiles_impl(tqr_plan h) {
    NvtxRange nvtx_("tqr_factor_tiles (a2-a7)");
    if (!h) return TQR_ERR_ARG;
    if (h->poisoned) return fail(h, TQR_ERR_STATE, "plan poisoned by an earlier CUDA/NCCL failure");
    if (h->ipc_mode && !h->ipc_connected) return fail(h, TQR_ERR_STATE, "IPC plan not connected (tqr_ipc_connect)");
    if (h->rs) return rs_factor(h);
    const int p = h->p, q = h->q, nb = h->nb, ib = h->ib;
    // bulk-update streams: round-robin (column lc on stream lc % S) for resident data; a streamed
    // factor maps contiguous chunks of columns to streams instead, so the early chunks run through
    // their steps while later columns are still being copied in (round-robin would block every
    // stream's step-1 launch behind its last column's load)
    const int S = h->streamed ? h->nstreams_io : h->nstreams;
    const int64_t tile = (int64_t)nb * nb, tsz = (int64_t)ib * nb, colsz = (int64_t)p * tile, vt = h->vt;
    const size_t es = h->es;
    const unsigned epoch0 = h->epoch;
    h->epoch += (unsigned)q + 1;
    h->factored = false;
    h->fact_gen += 1;
    // order all owner streams after whatever ran before (load, previous calls)
    for (auto& o : h->owners) {
        CUDA_TRY(h, cudaSetDevice(o.dev));
        CUDA_TRY(h, cudaStreamSynchronize(o.s_upd));
        if (h->profile) {
            for (auto& v : o.tm_used) std::fill(v.begin(), v.end(), 0);
            std::fill(o.tp_used.begin(), o.tp_used.end(), 0);
            std::fill(o.tb_used.begin(), o.tb_used.end(), 0);
            CUDA_TRY(h, cudaEventRecord(o.tref[0], o.s_panel));
        }
    }
    auto stream_of = [&](int lc, int nloc) -> int {
        return h->streamed ? (int)(((int64_t)lc * S) / nloc) : lc % S;
    };
    auto wait_all_u = [&](Owner& D, cudaStream_t st, int kk) -> tqr_status {
        for (int u = 0; u < S; ++u) CUDA_TRY(h, cudaStreamWaitEvent(st, D.ev_u[u][kk], 0));
        return TQR_OK;
    };
    // does rank / owner d hold a column > k (i.e. receive panel k)?
    auto needs = [&](int d, int k) {
        for (int j = k + 1; j < q; ++j) if (h->owner_of[j] == d) return true;
        return false;
    };
    auto emit = [&](int op, int k, int i, int j, int root) { h->issued.insert(h->issued.end(), {op, k, i, j, root}); };
    // The executor consumes the host-side DAG schedule (tqr_schedule: PANEL, BCAST, UPDATE records
    // per step), all owners' records for an in-process plan, this rank's for a multi-process one.
    std::vector<int32_t> sched;
    build_schedule(q, h->owner_of, h->multiproc() ? h->rank : -1, sched);
    h->issued.clear();
    const size_t nrec = sched.size() / 5;
    size_t pos = 0;
    while (pos < nrec) {
        const int op = sched[5 * pos], k = sched[5 * pos + 1];
        const int ok = h->owner_of[k];
        NvtxRange nvtx_op(op == 0 ? "PANEL(%d)" : (op == 1 ? "BCAST(%d)" : "UPDATE(%d)"), k);
        Owner* O = h->local(ok);
        if (op == 0) {
            // ---- PANEL(k)
            ++pos;
            if (!O) return fail(h, TQR_ERR_STATE, "schedule: PANEL(%d) of a remote owner", k);
            CUDA_TRY(h, cudaSetDevice(O->dev));
            if (k > 0 && !h->lookahead) { tqr_status st = wait_all_u(*O, O->s_panel, k - 1); if (st) return st; }
            if (h->streamed) CUDA_TRY(h, cudaStreamWaitEvent(O->s_panel, O->ev_load[O->lidx[k]], 0));
            // every prerequisite of PANEL(k) done: a remote lookahead trailing it may start spinning
            if (h->la_remote) CUDA_TRY(h, cudaEventRecord(O->ev_prepanel[k], O->s_panel));
            if (h->profile) CUDA_TRY(h, cudaEventRecord(O->tp0[k], O->s_panel));
            tqr_status st = launch_panel_step(h, *O, k, epoch0 + (unsigned)k + 1);
            if (st) return st;
            if (h->profile) { CUDA_TRY(h, cudaEventRecord(O->tp1[k], O->s_panel)); O->tp_used[k] = 1; }
            CUDA_TRY(h, cudaEventRecord(O->ev_panel[k], O->s_panel));
            emit(0, k, k, k, ok);
            if (h->streamed) {
                // column k is final once PANEL(k) is done (later steps touch columns > k only, and
                // updates read the reflectors from the stage images): a8 + D2H on the I/O stream
                const int lc = O->lidx[k];
                void* slab = h->at(O->io, (int64_t)lc * h->m * nb);
                CUDA_TRY(h, cudaStreamWaitEvent(O->s_io, O->ev_panel[k], 0));
                CUDA_TRY(h, from_tiles(h, slab, h->m, h->m * nb, h->at(O->tiles, lc * colsz), O->cols_dev + lc, 1,
                                       h->m, h->n, 1, O->s_io));
                CUDA_TRY(h, cudaMemcpy2DAsync(static_cast<char*>(h->sA) + (int64_t)k * nb * h->slda * es,
                                              h->slda * es, slab, h->m * es, h->m * es, group_cols(h, k),
                                              cudaMemcpyDefault, O->s_io));
                h->launches++;
            }
            continue;
        }
        if (op == 1) {
            // ---- BCAST(k): the reflector-tile images k..p-1, their T factors and the explicit V
            // (+ tree merge images / T) from owner(k) to every owner of a column > k
            ++pos;
            const int slot = k & 1;
            if (h->nccl_mode) {
                Owner& R = h->owners[0];
                CUDA_TRY(h, cudaSetDevice(R.dev));
                const bool root = (ok == h->rank);
                if (root) CUDA_TRY(h, cudaStreamWaitEvent(R.s_comm, R.ev_panel[k], 0));
                if (!root && k >= 2) {
                    tqr_status st = wait_all_u(R, R.s_comm, k - 2);
                    if (st) return st;
                    CUDA_TRY(h, cudaStreamWaitEvent(R.s_comm, R.ev_look[k - 2], 0));
                }
                if (h->profile) { CUDA_TRY(h, cudaEventRecord(R.tb0[k], R.s_comm)); }
                PanelRefs b = root ? own_refs(h, R, R.lidx[k]) : recv_refs(h, R, slot);
                const ncclDataType_t dt = h->f32() ? ncclFloat32 : ncclFloat64;
                void* bv = h->at(b.V, k * vt);
                void* bt = h->at(b.T, k * tsz);
                NCCL_TRY(h, h->nccl->GroupStart());
                NCCL_TRY(h, h->nccl->Broadcast(bv, bv, (size_t)(p - k) * vt, dt, ok, h->comm, R.s_comm));
                NCCL_TRY(h, h->nccl->Broadcast(bt, bt, (size_t)(p - k) * tsz, dt, ok, h->comm, R.s_comm));
                NCCL_TRY(h, h->nccl->Broadcast(b.Vexp, b.Vexp, (size_t)vt, dt, ok, h->comm, R.s_comm));
                if (h->ndom(k) > 1) {
                    const size_t D = h->ndom(k);
                    NCCL_TRY(h, h->nccl->Broadcast(b.M, b.M, D * vt, dt, ok, h->comm, R.s_comm));
                    NCCL_TRY(h, h->nccl->Broadcast(b.MT, b.MT, D * tsz, dt, ok, h->comm, R.s_comm));
                }
                NCCL_TRY(h, h->nccl->GroupEnd());
                CUDA_TRY(h, cudaEventRecord(R.ev_recv[k], R.s_comm));
                if (h->profile) {
                    CUDA_TRY(h, cudaEventRecord(R.tb1[k], R.s_comm));
                    R.tb_used[k] = 1;
                    h->stats[3].flops += (double)es * ((p - k) * (vt + tsz) + vt);
                }
            } else if (h->ipc_mode) {
                // root: copy into every receiver's IPC-mapped slot k%2 once that receiver has freed
                // it (its step k-2 updates are done), then raise the receiver's READY flag.
                // receiver: free the slot at the root, wait for READY.  All waits are on local flags.
                Owner& R = h->owners[0];
                CUDA_TRY(h, cudaSetDevice(R.dev));
                const uint64_t val = (uint64_t)epoch0 + 1 + k;
                if (ok == h->rank) {
                    CUDA_TRY(h, cudaStreamWaitEvent(R.s_comm, R.ev_panel[k], 0));
                    if (h->profile) CUDA_TRY(h, cudaEventRecord(R.tb0[k], R.s_comm));
                    const PanelRefs src = own_refs(h, R, R.lidx[k]);
                    std::vector<int> order;   // the lookahead owner (column k+1) first
                    if (k + 1 < q && h->owner_of[k + 1] != h->rank) order.push_back(h->owner_of[k + 1]);
                    for (int d = 0; d < h->world; ++d)
                        if (d != h->rank && (order.empty() || d != order[0])) order.push_back(d);
                    for (int d : order) {
                        if (!needs(d, k)) continue;
                        IpcPeer& P = h->peers[d];
                        CUDA_TRY(h, tqr::sig_wait_geq(R.s_comm, h->flags64 + F_FREED + 2 * d + slot, val));
                        if (h->la_remote && k + 1 < q && d == h->owner_of[k + 1]) {
                            // the lookahead owner: chunk c of tiles once PANEL(k) published its last tile
                            // (the TS chain publishes in order), then its chunk flag; it trails the panel
                            const int CH = h->la_chunk;
                            for (int t0 = k, c = 0; t0 < p; t0 += CH, ++c) {
                                const int t1 = std::min(p, t0 + CH);
                                CUDA_TRY(h, tqr::sig_wait_geq32(R.s_comm, R.flags + (int64_t)(t1 - 1) * (nb / ib) + nb / ib - 1,
                                                                epoch0 + (unsigned)k + 1));
                                CUDA_TRY(h, cudaMemcpyAsync(h->at(P.rb[slot][0], t0 * vt), h->at(src.V, t0 * vt),
                                                            es * (size_t)(t1 - t0) * vt, cudaMemcpyDefault, R.s_comm));
                                CUDA_TRY(h, cudaMemcpyAsync(h->at(P.rb[slot][1], t0 * tsz), h->at(src.T, t0 * tsz),
                                                            es * (size_t)(t1 - t0) * tsz, cudaMemcpyDefault, R.s_comm));
                                if (t0 == k)
                                    CUDA_TRY(h, cudaMemcpyAsync(P.rb[slot][2], src.Vexp, es * (size_t)vt, cudaMemcpyDefault,
                                                                R.s_comm));
                                CUDA_TRY(h, tqr::sig_write(R.s_comm, P.flags + F_CHUNK + slot * kMaxChunks + c, val));
                            }
                            CUDA_TRY(h, tqr::sig_write(R.s_comm, P.flags + F_READY + slot, val));
                            if (h->profile) h->stats[3].flops += (double)es * ((p - k) * (vt + tsz) + vt);
                            continue;
                        }
                        CUDA_TRY(h, cudaMemcpyAsync(h->at(P.rb[slot][0], k * vt), h->at(src.V, k * vt),
                                                    es * (size_t)(p - k) * vt, cudaMemcpyDefault, R.s_comm));
                        CUDA_TRY(h, cudaMemcpyAsync(h->at(P.rb[slot][1], k * tsz), h->at(src.T, k * tsz),
                                                    es * (size_t)(p - k) * tsz, cudaMemcpyDefault, R.s_comm));
                        CUDA_TRY(h, cudaMemcpyAsync(P.rb[slot][2], src.Vexp, es * (size_t)vt, cudaMemcpyDefault, R.s_comm));
                        if (h->ndom(k) > 1) {
                            const size_t nd = h->ndom(k);
                            CUDA_TRY(h, cudaMemcpyAsync(P.rb[slot][3], src.M, es * nd * vt, cudaMemcpyDefault, R.s_comm));
                            CUDA_TRY(h, cudaMemcpyAsync(P.rb[slot][4], src.MT, es * nd * tsz, cudaMemcpyDefault, R.s_comm));
                        }
                        CUDA_TRY(h, tqr::sig_write(R.s_comm, P.flags + F_READY + slot, val));
                        if (h->profile) h->stats[3].flops += (double)es * ((p - k) * (vt + tsz) + vt);
                    }
                    if (h->profile) { CUDA_TRY(h, cudaEventRecord(R.tb1[k], R.s_comm)); R.tb_used[k] = 1; }
                } else if (needs(h->rank, k)) {
                    if (k >= 2) {
                        tqr_status st = wait_all_u(R, R.s_comm, k - 2);
                        if (st) return st;
                        CUDA_TRY(h, cudaStreamWaitEvent(R.s_comm, R.ev_look[k - 2], 0));
                    }
                    CUDA_TRY(h, tqr::sig_write(R.s_comm, h->peers[ok].flags + F_FREED + 2 * h->rank + slot, val));
                    CUDA_TRY(h, tqr::sig_wait_geq(R.s_comm, h->flags64 + F_READY + slot, val));
                    CUDA_TRY(h, cudaEventRecord(R.ev_recv[k], R.s_comm));
                }
            } else {
                for (auto& D : h->owners) {
                    if (D.id == ok || !needs(D.id, k)) continue;
                    CUDA_TRY(h, cudaSetDevice(D.dev));
                    const bool trail = h->la_remote && k + 1 < q && D.id == h->owner_of[k + 1];
                    if (!trail) CUDA_TRY(h, cudaStreamWaitEvent(D.s_comm, O->ev_panel[k], 0));
                    if (k >= 2) {
                        tqr_status st = wait_all_u(D, D.s_comm, k - 2);
                        if (st) return st;
                        CUDA_TRY(h, cudaStreamWaitEvent(D.s_comm, D.ev_look[k - 2], 0));
                    }
                    if (h->profile) CUDA_TRY(h, cudaEventRecord(D.tb0[k], D.s_comm));
                    const PanelRefs src = own_refs(h, *O, O->lidx[k]);
                    if (trail) {
                        // the lookahead owner: chunks of tiles as PANEL(k) publishes them (stream wait on
                        // the panel's own flags), a chunk flag after each; the lookahead trails them
                        CUDA_TRY(h, cudaStreamWaitEvent(D.s_comm, O->ev_prepanel[k], 0));
                        const int CH = h->la_chunk;
                        const uint64_t val = (uint64_t)epoch0 + 1 + k;
                        for (int t0 = k, c = 0; t0 < p; t0 += CH, ++c) {
                            const int t1 = std::min(p, t0 + CH);
                            CUDA_TRY(h, tqr::sig_wait_geq32(D.s_comm, O->flags + (int64_t)(t1 - 1) * (nb / ib) + nb / ib - 1,
                                                            epoch0 + (unsigned)k + 1));
                            CUDA_TRY(h, cudaMemcpyPeerAsync(h->at(D.rb_tiles[slot], t0 * vt), D.dev, h->at(src.V, t0 * vt),
                                                            O->dev, es * (size_t)(t1 - t0) * vt, D.s_comm));
                            CUDA_TRY(h, cudaMemcpyPeerAsync(h->at(D.rb_T[slot], t0 * tsz), D.dev, h->at(src.T, t0 * tsz),
                                                            O->dev, es * (size_t)(t1 - t0) * tsz, D.s_comm));
                            if (t0 == k)
                                CUDA_TRY(h, cudaMemcpyPeerAsync(D.rb_V[slot], D.dev, src.Vexp, O->dev, es * (size_t)vt,
                                                                D.s_comm));
                            CUDA_TRY(h, tqr::sig_write(D.s_comm, reinterpret_cast<uint64_t*>(D.cflg) + slot * kMaxChunks + c, val));
                        }
                        CUDA_TRY(h, cudaEventRecord(D.ev_recv[k], D.s_comm));
                        if (h->profile) {
                            CUDA_TRY(h, cudaEventRecord(D.tb1[k], D.s_comm));
                            D.tb_used[k] = 1;
                            h->stats[3].flops += (double)es * ((p - k) * (vt + tsz) + vt);
                        }
                        continue;
                    }
                    CUDA_TRY(h, cudaMemcpyPeerAsync(h->at(D.rb_tiles[slot], k * vt), D.dev, h->at(src.V, k * vt), O->dev,
                                                    es * (size_t)(p - k) * vt, D.s_comm));
                    CUDA_TRY(h, cudaMemcpyPeerAsync(h->at(D.rb_T[slot], k * tsz), D.dev, h->at(src.T, k * tsz), O->dev,
                                                    es * (size_t)(p - k) * tsz, D.s_comm));
                    CUDA_TRY(h, cudaMemcpyPeerAsync(D.rb_V[slot], D.dev, src.Vexp, O->dev, es * (size_t)vt, D.s_comm));
                    if (h->ndom(k) > 1) {
                        const size_t nd = h->ndom(k);
                        CUDA_TRY(h, cudaMemcpyPeerAsync(D.rb_M[slot], D.dev, src.M, O->dev, es * nd * vt, D.s_comm));
                        CUDA_TRY(h, cudaMemcpyPeerAsync(D.rb_MT[slot], D.dev, src.MT, O->dev, es * nd * tsz, D.s_comm));
                    }
                    CUDA_TRY(h, cudaEventRecord(D.ev_recv[k], D.s_comm));
                    if (h->profile) {
                        CUDA_TRY(h, cudaEventRecord(D.tb1[k], D.s_comm));
                        D.tb_used[k] = 1;
                        h->stats[3].flops += (double)es * ((p - k) * (vt + tsz) + vt);
                    }
                }
            }
            emit(1, k, k, k, ok);
            continue;
        }
        // ---- UPDATE(k): the run of UPDATE records of step k (one per column j > k of a local owner)
        size_t end = pos;
        int64_t nsched = 0;
        while (end < nrec && sched[5 * end] == 2 && sched[5 * end + 1] == k) { ++end; ++nsched; }
        pos = end;
        int64_t nlocal = 0;
        for (auto& D : h->owners) {
            CUDA_TRY(h, cudaSetDevice(D.dev));
            const bool mine = (D.id == ok);
            const int slot = k & 1;
            const PanelRefs r = mine ? own_refs(h, D, D.lidx[k]) : recv_refs(h, D, slot);
            cudaEvent_t ready = mine ? D.ev_panel[k] : D.ev_recv[k];
            // local columns j > k form a suffix [first, ncols) of D.cols
            int first = (int)(std::upper_bound(D.cols.begin(), D.cols.end(), k) - D.cols.begin());
            const int nloc = (int)D.cols.size();
            nlocal += nloc - first;
            const bool la = h->lookahead && first < nloc && D.cols[first] == k + 1;
            if (la) {
                // lookahead: column k+1 first, on a high-priority stream.  FP64 flat panel of this
                // owner: the update runs beside PANEL(k) (already enqueued, so its CTAs are
                // dispatched first) and waits per reflector tile on the panel's flags; otherwise it
                // follows the whole panel (or the broadcast) on the panel stream.
                // (not with logical owners: several owners' lookaheads could then spin on one GPU)
                // logical owners share one GPU: the local overlap there too, behind the pre-panel event
                // (at most one lookahead spins at a time, as for the remote trailing one)
                const bool ovl = mine && h->la_overlap && h->la_fits && (!h->logical || h->la_remote) && !h->f32() &&
                                 h->ndom(k) == 1;
                // remote panel: trail its chunks (chunk flags of the receive slot) instead of the whole panel
                const bool rtrail = !mine && h->la_remote && !h->f32() && h->ndom(k) == 1;
                cudaStream_t sl = (ovl || rtrail) ? D.s_look : D.s_panel;
                if (!ovl && !rtrail) CUDA_TRY(h, cudaStreamWaitEvent(sl, ready, 0));
                if ((rtrail && O) || (ovl && h->logical))
                    CUDA_TRY(h, cudaStreamWaitEvent(sl, O->ev_prepanel[k], 0));   // in-process root
                if (k >= 1) CUDA_TRY(h, cudaStreamWaitEvent(sl, D.ev_u[stream_of(first, (int)D.cols.size())][k - 1], 0));
                if (k == 0 && h->streamed) CUDA_TRY(h, cudaStreamWaitEvent(sl, D.ev_load[first], 0));
                const int wl = w_look(h);
                const unsigned long long* cf = nullptr;
                if (rtrail)
                    cf = h->ipc_mode ? reinterpret_cast<const unsigned long long*>(h->flags64 + F_CHUNK + slot * kMaxChunks)
                                     : D.cflg + slot * kMaxChunks;
                CUDA_TRY(h, update(h, r, D.tiles, colsz, tile, nb, first, 1, k, wl, nb / wl, true, sl,
                                   &h->launches, ovl ? D.flags : nullptr, epoch0 + (unsigned)k + 1,
                                   cf, (unsigned long long)epoch0 + 1 + k, h->la_chunk));
                emit(2, k, k, D.cols[first], ok);
                if (ovl || rtrail) {   // PANEL(k+1) (panel stream) after the lookahead
                    CUDA_TRY(h, cudaEventRecord(D.ev_look[k], sl));
                    CUDA_TRY(h, cudaStreamWaitEvent(D.s_panel, D.ev_look[k], 0));
                }
                first += 1;
            }
            CUDA_TRY(h, cudaEventRecord(D.ev_look[k], D.s_panel));
            // bulk: columns lc in [first, nloc) with lc % S == u on stream u (stream order chains
            // column lc's step k-1 -> k updates; steps overlap across streams)
            for (int uu = 0; uu < S; ++uu) {
                int g0, ng, gs;
                if (h->streamed) {   // chunk [lo, hi) of the local columns
                    const int lo = (int)(((int64_t)uu * nloc + S - 1) / S), hi = (int)(((int64_t)(uu + 1) * nloc + S - 1) / S);
                    g0 = std::max(lo, first);
                    ng = std::max(0, hi - g0);
                    gs = 1;
                } else {
                    g0 = first + ((uu - first % S) + S) % S;
                    ng = (g0 < nloc) ? (nloc - g0 + S - 1) / S : 0;
                    gs = S;
                }
                cudaStream_t su = D.s_u[uu];
                if (h->cp_probe && ng > 0) {   // keep the dependency structure, skip the work
                    CUDA_TRY(h, cudaStreamWaitEvent(su, ready, 0));
                } else if (ng > 0) {
                    CUDA_TRY(h, cudaStreamWaitEvent(su, ready, 0));
                    if (h->profile) CUDA_TRY(h, cudaEventRecord(D.tm0[uu][k], su));
                    const int wb = w_bulk(h);
                    if (k == 0 && h->streamed) {
                        // step 0 of a streamed factor: the chunk's columns load in order, so waiting
                        // for its last one covers them all; one launch keeps the chunk's columns
                        // concurrent (per-column launches on one stream would run one at a time)
                        CUDA_TRY(h, cudaStreamWaitEvent(su, D.ev_load[g0 + (ng - 1) * gs], 0));
                    }
                    CUDA_TRY(h, update(h, r, D.tiles, colsz, tile, nb, g0, gs, k, wb, ng * (nb / wb), true, su,
                                       &h->launches));
                    if (h->profile) {
                        CUDA_TRY(h, cudaEventRecord(D.tm1[uu][k], su));
                        D.tm_used[uu][k] = 1;
                        h->stats[0].flops += flops_update(h, k, ng);
                        h->stats[0].count += 1;
                    }
                }
                for (int c = 0; c < ng; ++c) emit(2, k, k, D.cols[g0 + c * gs], ok);
                CUDA_TRY(h, cudaEventRecord(D.ev_u[uu][k], su));
            }
        }
        if (nlocal != nsched)
            return fail(h, TQR_ERR_STATE, "schedule: step %d lists %lld updates, %lld local columns", k,
                        (long long)nsched, (long long)nlocal);
    }
    tqr_status st = sync_all(h);
    if (st) return st;
    if (h->profile) {
        for (auto& o : h->owners) {
            CUDA_TRY(h, cudaSetDevice(o.dev));
            std::vector<std::pair<double, double>> iv, ip, ib_;
            for (int k = 0; k < q; ++k) {
                float a = 0.f, b = 0.f;
                for (int uu = 0; uu < S; ++uu)
                    if (o.tm_used[uu][k]) {
                        CUDA_TRY(h, cudaEventElapsedTime(&a, o.tref[0], o.tm0[uu][k]));
                        CUDA_TRY(h, cudaEventElapsedTime(&b, o.tref[0], o.tm1[uu][k]));
                        iv.push_back({a, b});
                    }
                if (o.tp_used[k]) {
                    CUDA_TRY(h, cudaEventElapsedTime(&a, o.tref[0], o.tp0[k]));
                    CUDA_TRY(h, cudaEventElapsedTime(&b, o.tref[0], o.tp1[k]));
                    ip.push_back({a, b});
                    h->stats[1].count += 1;
                    h->stats[1].flops += flops_panel(h, k);
                }
                if (o.tb_used[k] && o.dev == h->owners[0].dev) {
                    CUDA_TRY(h, cudaEventElapsedTime(&a, o.tref[0], o.tb0[k]));
                    CUDA_TRY(h, cudaEventElapsedTime(&b, o.tref[0], o.tb1[k]));
                    ib_.push_back({a, b});
                    h->stats[3].count += 1;
                }
            }
            h->stats[0].ms += union_ms(iv);
            h->stats[1].ms += union_ms(ip);
            h->stats[3].ms += union_ms(ib_);
        }
    }
    if (h->ipc_mode) {
        // next factorization: my receive slots 0 / 1 are free for its steps 0 / 1 (at every root);
        // this factorization is complete on this rank (apply/solve replication may read it)
        Owner& R = h->owners[0];
        CUDA_TRY(h, cudaSetDevice(R.dev));
        h->fact_id = (uint64_t)epoch0 + 1;
        for (int d = 0; d < h->world; ++d) {
            if (d == h->rank) continue;
            for (int sl = 0; sl < 2; ++sl)
                CUDA_TRY(h, tqr::sig_write(R.s_comm, h->peers[d].flags + F_FREED + 2 * h->rank + sl,
                                           (uint64_t)h->epoch + 1 + sl));
            CUDA_TRY(h, tqr::sig_write(R.s_comm, h->peers[d].flags + F_DONE + h->rank, h->fact_id));
        }
        { tqr_status ws = wait_stream(h, R.s_comm); if (ws) return ws; }
    }
    h->factored = true;
    return TQR_OK;
}

// ------------------------------------------------------------------ a8: R out
static tqr_status tqr_store_r_impl(tqr_plan h, void* A, int64_t lda) {
    NvtxRange nvtx_("tqr_store_r (a8)");
    if (!h) return TQR_ERR_ARG;
    if (h->poisoned) return fail(h, TQR_ERR_STATE, "plan poisoned by an earlier CUDA/NCCL failure");
    if (!h->factored) return fail(h, TQR_ERR_STATE, "store_r before factor");
    if (!A || lda < h->m) return fail(h, TQR_ERR_ARG, "store_r: A is NULL or lda < m");
    if (h->rs) return rs_store(h, A, lda);
    const PtrInfo pi = classify(A);
    const int64_t nb = h->nb, es = h->es;
    { tqr_status st0 = sync_entry(h, pi); if (st0) return st0; }
    for (auto& o : h->owners) {
        if (o.cols.empty()) continue;
        CUDA_TRY(h, cudaSetDevice(o.dev));
        const int nc = (int)o.cols.size();
        if (h->profile) CUDA_TRY(h, cudaEventRecord(o.tl[2], o.s_upd));
        if (pi.kind == Mem::Device && pi.dev == o.dev) {
            CUDA_TRY(h, from_tiles(h, A, lda, nb * lda, o.tiles, o.cols_dev, nc, h->m, h->n, 0, o.s_upd));
            h->launches++;
        } else {
            tqr_status st = ensure_io(h, o);
            if (st) return st;
            CUDA_TRY(h, from_tiles(h, o.io, h->m, h->m * nb, o.tiles, o.cols_dev, nc, h->m, h->n, 1, o.s_upd));
            h->launches++;
            for (int lc = 0; lc < nc; ++lc) {
                const int64_t j = o.cols[lc];
                CUDA_TRY(h, cudaMemcpy2DAsync(static_cast<char*>(A) + j * nb * lda * es, lda * es,
                                              h->at(o.io, (int64_t)lc * h->m * nb), h->m * es, h->m * es,
                                              group_cols(h, j), cudaMemcpyDefault, o.s_upd));
            }
        }
        if (h->profile) CUDA_TRY(h, cudaEventRecord(o.tl[3], o.s_upd));
    }
    tqr_status st = sync_all(h);
    if (st) return st;
    return layout_stat(h, 2);
}

// Streamed factor of a single tile column in tree mode (C4-like, one owner, one CTA per domain):
// the rows arrive in NC chunks of whole TS domains on the I/O stream (H2D + a1 per chunk); each
// chunk's domains start on their own stream as soon as the chunk is resident; the rows >= nb of a
// chunk are zero in the result, so they are written back (zeros, device -> host on the comm
// stream, full duplex with the loads) as soon as the chunk has been read; after the merges only
// the first tile row (R) is copied out.
namespace {
tqr_status factor_streamed_tall(tqr_plan h, void* A, int64_t lda) {
    Owner& O = h->owners[0];
    const int nb = h->nb, p = h->p, L = h->tree_L, D = h->ndom(0);
    const int64_t m = h->m, es = h->es, tile = (int64_t)nb * nb, colsz = (int64_t)p * tile;
    const int NC = std::min(D, 8);
    CUDA_TRY(h, cudaSetDevice(O.dev));
    tqr_status st = ensure_io(h, O);
    if (st) return st;
    auto mk = [&](std::vector<cudaEvent_t>& v) -> tqr_status {
        while ((int)v.size() < NC) {
            cudaEvent_t e;
            CUDA_TRY(h, cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
            v.push_back(e);
        }
        return TQR_OK;
    };
    if ((st = mk(O.ev_chunk)) || (st = mk(O.ev_dom))) return st;
    const unsigned epoch0 = h->epoch;
    h->epoch += 2;
    h->factored = false;
    double* col = h->at<double>(O.tiles, 0);
    const PanelRefs r = own_refs(h, O, 0);
    for (int c = 0; c < NC; ++c) {
        const int d0 = (int)((int64_t)c * D / NC), d1 = (int)((int64_t)(c + 1) * D / NC);
        const int t0 = d0 * L, t1 = std::min(d1 * L, p);
        const int64_t r0 = (int64_t)t0 * nb, r1 = std::min<int64_t>((int64_t)t1 * nb, m);
        void* slab = h->at(O.io, r0);
        if (r1 > r0) {
            CUDA_TRY(h, cudaMemcpy2DAsync(slab, m * es, static_cast<const char*>(A) + r0 * es, lda * es, (r1 - r0) * es,
                                          h->n, cudaMemcpyDefault, O.s_io));
        }
        CUDA_TRY(h, tqr::launch_to_tiles<double>((const double*)slab, m, m * nb, col + (int64_t)t0 * tile, O.cols_dev,
                                                 1, 1, colsz, nb, t1 - t0, std::max<int64_t>(r1 - r0, 0), h->n, O.s_io));
        CUDA_TRY(h, cudaEventRecord(O.ev_chunk[c], O.s_io));
        cudaStream_t sd = O.s_u[c % O.s_u.size()];
        CUDA_TRY(h, cudaStreamWaitEvent(sd, O.ev_chunk[c], 0));
        tqr::DomainArgs da{col, (double*)r.T, (double*)r.V, (double*)r.Vexp, 0, p, L};
        da.dom0 = d0;
        CUDA_TRY(h, tqr::launch_domains(nb, h->ib, da, d1 - d0, sd));
        CUDA_TRY(h, cudaEventRecord(O.ev_dom[c], sd));
        // result rows [max(r0, nb), r1) are zero: the slab rows were consumed by a1 -> zero them
        // on the device and write them back while later chunks load
        const int64_t z0 = std::max<int64_t>(r0, nb);
        if (r1 > z0) {
            CUDA_TRY(h, cudaStreamWaitEvent(O.s_comm, O.ev_chunk[c], 0));
            void* zs = h->at(O.io, z0);
            CUDA_TRY(h, cudaMemset2DAsync(zs, m * es, 0, (r1 - z0) * es, h->n, O.s_comm));
            CUDA_TRY(h, cudaMemcpy2DAsync(static_cast<char*>(A) + z0 * es, lda * es, zs, m * es, (r1 - z0) * es, h->n,
                                          cudaMemcpyDefault, O.s_comm));
        }
        h->launches += 2;
    }
    for (int c = 0; c < NC; ++c) CUDA_TRY(h, cudaStreamWaitEvent(O.s_panel, O.ev_dom[c], 0));
    h->domains_done = true;
    st = launch_panel_step(h, O, 0, epoch0 + 1);
    h->domains_done = false;
    if (st) return st;
    // R: the first tile row only (a8 for rows 0..min(nb, m)), after the merges
    const int64_t rr = std::min<int64_t>(nb, m);
    CUDA_TRY(h, tqr::launch_from_tiles<double>((double*)O.io, m, m * nb, col, O.cols_dev, 1, colsz, nb, rr, h->n, 1,
                                               O.s_panel));
    CUDA_TRY(h, cudaMemcpy2DAsync(A, lda * es, O.io, m * es, rr * es, h->n, cudaMemcpyDefault, O.s_panel));
    h->launches++;
    st = sync_all(h);
    if (st) return st;
    h->factored = true;
    h->fact_gen += 1;
    return TQR_OK;
}
}  // namespace

// A not resident on the owners' devices (host memory, or another GPU): the I/O is pipelined with
// the factorization -- column tile j is copied in and converted (a1) on the owner's I/O stream,
// PANEL(j) and the step-0 update of column j wait only for column j, and R of column k (a8) is
// copied out as soon as PANEL(k) completes, so only the first column's load and the last
// column's store are exposed.  A is in place (the columns being read are never the ones written).
static tqr_status tqr_factor_impl(tqr_plan h, void* A, int64_t lda) {
    NvtxRange nvtx_("tqr_factor");
    if (!h) return TQR_ERR_ARG;
    if (h->poisoned) return fail(h, TQR_ERR_STATE, "plan poisoned by an earlier CUDA/NCCL failure");
    if (!A || lda < h->m) return fail(h, TQR_ERR_ARG, "factor: A is NULL or lda < m");
    if (h->rs) {
        tqr_status st = rs_load(h, A, lda);
        if (!st) st = rs_factor(h);
        if (!st) st = rs_store(h, A, lda);
        return st;
    }
    const PtrInfo pi = classify(A);
    bool resident = true;
    for (auto& o : h->owners)
        if (!o.cols.empty() && !(pi.kind == Mem::Device && pi.dev == o.dev)) resident = false;
    if (resident || getenv("TQR_NO_STREAMED_IO")) {
        tqr_status st = tqr_load(h, A, lda);
        if (st) return st;
        st = tqr_factor_tiles(h);
        if (st) return st;
        return tqr_store_r(h, A, lda);
    }
    const int64_t nb = h->nb, es = h->es, colsz = (int64_t)h->p * nb * nb;
    h->factored = false;
    { tqr_status st0 = sync_entry(h, pi); if (st0) return st0; }
    if (h->q == 1 && h->tree_L > 0 && h->tree_one_cta && h->owners.size() == 1 && !h->multiproc() && !h->f32() &&
        h->ndom(0) > 1 && !getenv("TQR_NO_STREAMED_TALL"))
        return factor_streamed_tall(h, A, lda);
    for (auto& o : h->owners) {
        if (o.cols.empty()) continue;
        CUDA_TRY(h, cudaSetDevice(o.dev));
        tqr_status st = ensure_io(h, o);
        if (st) return st;
        for (int lc = 0; lc < (int)o.cols.size(); ++lc) {
            const int64_t j = o.cols[lc];
            void* slab = h->at(o.io, (int64_t)lc * h->m * nb);
            CUDA_TRY(h, cudaMemcpy2DAsync(slab, h->m * es, static_cast<const char*>(A) + j * nb * lda * es, lda * es,
                                          h->m * es, group_cols(h, j), cudaMemcpyDefault, o.s_io));
            CUDA_TRY(h, to_tiles(h, slab, h->m, h->m * nb, h->at(o.tiles, lc * colsz), o.cols_dev + lc, 1, 1, o.s_io));
            CUDA_TRY(h, cudaEventRecord(o.ev_load[lc], o.s_io));
            h->launches++;
        }
    }
    h->streamed = true;
    h->sA = A;
    h->slda = lda;
    tqr_status st = tqr_factor_tiles(h);
    h->streamed = false;
    h->sA = nullptr;
    if (st) sync_all(h);
    return st;
}

// ------------------------------------------------------------------ apply Q^T / Q, solve
// Owners on several GPUs, or several processes: apply/solve run on a single-owner replica of the
// factorization on this process's device, gathered once per factorization (peer copies / IPC
// pulls from the owners' memory / ncclBroadcast from each column's owner).
static bool needs_replica(tqr_plan h) {
    if (h->multiproc()) return true;
    if (const char* e = getenv("TQR_FORCE_REPLICA")) if (atoi(e) != 0 && h->owners.size() > 1) return true;
    for (auto& o : h->owners)
        if (o.dev != h->owners[0].dev) return true;
    return false;
}

static tqr_status ensure_replica(tqr_plan h) {
    if (h->rep && h->rep_gen == h->fact_gen) return TQR_OK;
    const int dev = h->owners[0].dev;
    CUDA_TRY(h, cudaSetDevice(dev));
    if (!h->rep) {
        tqr_options o{};
        o.logical_devices = 1;
        o.no_lookahead = 1;
        o.row_split = -1;
        o.tree_domain = h->tree_L > 0 ? h->tree_L : -1;
        o.tree_group = h->tree_G > 1 ? h->tree_G : -1;
        tqr_status st = tqr_create_ex(h->m, h->n, h->nb, h->ib, h->dtype, 1, nullptr, 0, &o, &h->rep);
        if (st) return fail(h, st, "apply/solve replica: %s", g_create_error.c_str());
        if (h->rep->tree_L != h->tree_L || h->rep->tree_G != h->tree_G || h->rep->dmax != h->dmax)
            return fail(h, TQR_ERR_STATE, "apply/solve replica: elimination tree mismatch");
    }
    tqr_plan r = h->rep;
    Owner& RO = r->owners[0];                       // owns every column, lidx[j] == j
    const int64_t p = h->p, tile = (int64_t)h->nb * h->nb, tsz = (int64_t)h->ib * h->nb, vt = h->vt;
    const int64_t dm = h->tree_L > 0 ? h->dmax : 0;
    const int64_t sz[6] = {p * tile, p * vt, p * tsz, vt, dm * vt, dm * tsz};   // per column, elements
    void* dst_base[6] = {RO.tiles, RO.Vimg, RO.T, RO.Vexp, RO.Mimg, RO.MT};
    cudaStream_t s = RO.s_upd;
    const size_t es = h->es;
    if (h->nccl_mode) NCCL_TRY(h, h->nccl->GroupStart());
    for (int j = 0; j < h->q; ++j) {
        const int o = h->owner_of[j];
        int lc = 0;                                 // j's index among its owner's columns
        for (int jj = 0; jj < j; ++jj) lc += (h->owner_of[jj] == o);
        const bool local = !h->multiproc() || o == h->rank;
        Owner* O = local ? h->local(o) : nullptr;
        void* src_base[6] = {nullptr};
        int src_dev = dev;
        if (local) {
            void* b[6] = {O->tiles, O->Vimg, O->T, O->Vexp, O->Mimg, O->MT};
            for (int f = 0; f < 6; ++f) src_base[f] = b[f];
            src_dev = O->dev;
        } else if (h->ipc_mode) {
            for (int f = 0; f < 6; ++f) src_base[f] = h->peers[o].st[f];
            src_dev = h->peers[o].dev;
            CUDA_TRY(h, tqr::sig_wait_geq(s, h->flags64 + F_DONE + o, h->fact_id));
        }
        for (int f = 0; f < 6; ++f) {
            if (sz[f] == 0) continue;
            void* dst = h->at(dst_base[f], (int64_t)j * sz[f]);
            if (h->nccl_mode) {
                const void* sb = local ? h->at(src_base[f], (int64_t)lc * sz[f]) : dst;
                NCCL_TRY(h, h->nccl->Broadcast(sb, dst, (size_t)sz[f], h->f32() ? ncclFloat32 : ncclFloat64, o, h->comm, s));
            } else {
                CUDA_TRY(h, cudaMemcpyPeerAsync(dst, dev, h->at(src_base[f], (int64_t)lc * sz[f]), src_dev, es * sz[f], s));
            }
        }
    }
    if (h->nccl_mode) NCCL_TRY(h, h->nccl->GroupEnd());
    { tqr_status ws = wait_stream(h, s); if (ws) return ws; }
    r->factored = true;
    h->rep_gen = h->fact_gen;
    return TQR_OK;
}

// IPC collective epilogue of apply / solve: return only when every rank has finished reading the
// owners' storage (so no rank's next factor overwrites reflectors a peer is still pulling).
static tqr_status ipc_apply_barrier(tqr_plan h) {
    if (!h->ipc_mode) return TQR_OK;
    h->apply_seq += 1;
    cudaStream_t s = h->owners[0].s_comm;
    CUDA_TRY(h, cudaSetDevice(h->owners[0].dev));
    for (int d = 0; d < h->world; ++d)
        if (d != h->rank) CUDA_TRY(h, tqr::sig_write(s, h->peers[d].flags + F_APPLIED + h->rank, h->apply_seq));
    for (int d = 0; d < h->world; ++d)
        if (d != h->rank) CUDA_TRY(h, tqr::sig_wait_geq(s, h->flags64 + F_APPLIED + d, h->apply_seq));
    { tqr_status ws = wait_stream(h, s); if (ws) return ws; }
    return TQR_OK;
}

static tqr_status single_device(tqr_plan h, int* dev) {
    *dev = h->owners[0].dev;
    return TQR_OK;
}

// Row split (single process): Q = diag(Q_g) E Q_top, where E embeds the stacked first nb rows of
// every owner's block (the rows of R_g) into the stage-2 stack.  Q^T B: every block B_g <- Q_g^T B_g,
// gather the blocks' first nb rows into the stack, stack <- Q_top^T stack, scatter back.  Q B: the
// reverse.  Stack rows past an owner's block (rows_g < nb) are zero rows of the stacked R and stay
// zero under Q_top, so they are dropped.  solve_ls: the stack is solved by the stage-2 plan (its R is
// the final R) and X comes from the stack's first n rows.
static tqr_status rs_apply(tqr_plan h, char trans, void* B, int64_t ldb, int64_t nrhs, bool solve) {
    if (h->multiproc()) return fail(h, TQR_ERR_UNSUPPORTED, "apply/solve: multi-process row-split plans keep Q distributed");
    const bool fwd = solve || trans == 'T' || trans == 't';
    const int G = h->ndev, nb = h->nb;
    const int64_t es = h->es, ls = (int64_t)G * nb;
    CUDA_TRY(h, cudaSetDevice(h->top_dev));
    if ((size_t)(ls * nrhs) > h->bw_elems) {
        if (h->bw) cudaFree(h->bw);
        h->bw = nullptr;
        h->bw_elems = 0;
        CUDA_TRY(h, cudaMalloc(&h->bw, (size_t)(ls * nrhs) * es));
        h->bw_elems = (size_t)(ls * nrhs);
    }
    auto kids_apply = [&](char tr) -> tqr_status {
        for (size_t i = 0; i < h->kids.size(); ++i) {
            CUDA_TRY(h, cudaSetDevice(h->kid_dev[i]));
            const int g = h->kid_owner[i];
            tqr_status st = tqr_apply_qt(h->kids[i], tr, static_cast<char*>(B) + h->rs_r0[g] * es, ldb, nrhs);
            if (st) return kid_fail(h, h->kids[i], st);
        }
        return TQR_OK;
    };
    auto gather = [&](bool in) -> tqr_status {
        CUDA_TRY(h, cudaSetDevice(h->top_dev));
        if (in) CUDA_TRY(h, cudaMemset(h->bw, 0, (size_t)(ls * nrhs) * es));
        for (int g = 0; g < G; ++g) {
            const int64_t rows = std::min<int64_t>(nb, h->rs_rows[g]);
            char* Bg = static_cast<char*>(B) + h->rs_r0[g] * es;
            char* Sg = static_cast<char*>(h->bw) + (int64_t)g * nb * es;
            if (in) CUDA_TRY(h, cudaMemcpy2D(Sg, ls * es, Bg, ldb * es, rows * es, nrhs, cudaMemcpyDefault));
            else CUDA_TRY(h, cudaMemcpy2D(Bg, ldb * es, Sg, ls * es, rows * es, nrhs, cudaMemcpyDefault));
        }
        return TQR_OK;
    };
    tqr_status st = TQR_OK;
    if (fwd) {
        if ((st = kids_apply('T')) || (st = gather(true))) return st;
        CUDA_TRY(h, cudaSetDevice(h->top_dev));
        st = solve ? tqr_solve_ls(h->top, h->bw, ls, nrhs) : tqr_apply_qt(h->top, 'T', h->bw, ls, nrhs);
        if (st) return kid_fail(h, h->top, st);
        if (solve) {
            CUDA_TRY(h, cudaMemcpy2D(B, ldb * es, h->bw, ls * es, h->n * es, nrhs, cudaMemcpyDefault));
            return TQR_OK;
        }
        return gather(false);
    }
    if ((st = gather(true))) return st;
    CUDA_TRY(h, cudaSetDevice(h->top_dev));
    st = tqr_apply_qt(h->top, 'N', h->bw, ls, nrhs);
    if (st) return kid_fail(h, h->top, st);
    if ((st = gather(false))) return st;
    return kids_apply('N');
}

// Bw (mp x 32*nslices, ld ldw) <- Q^T Bw (forward over the panels) or Q Bw (reverse).
// FP64, one owner, flat tree: all q steps in one wavefront launch (step k+1's chain follows step
// k's tile by tile), otherwise one launch per step.
static tqr_status apply_device(tqr_plan h, char trans, void* Bw, int64_t ldw, int64_t nslices, cudaStream_t s) {
    const int q = h->q, nb = h->nb;
    const bool fwd = (trans == 'T' || trans == 't');
    if (!h->f32() && h->tree_L == 0 && h->owners.size() == 1 && q > 1 && !getenv("TQR_NO_WAVEFRONT_APPLY")) {
        Owner& O = h->owners[0];
        const size_t need = (size_t)q * nslices;
        if (need > h->prog_n) {
            if (h->prog) cudaFree(h->prog);
            h->prog = nullptr;
            h->prog_n = 0;
            CUDA_TRY(h, cudaMalloc(&h->prog, need * sizeof(unsigned)));
            h->prog_n = need;
        }
        CUDA_TRY(h, cudaMemsetAsync(h->prog, 0, need * sizeof(unsigned), s));
        const int k0 = fwd ? 0 : q - 1;
        const PanelRefs r = own_refs(h, O, O.lidx[k0]);
        const int64_t p = h->p;
        tqr::UpdateArgs u;
        u.V = (const double*)r.V; u.T = (const double*)r.T; u.Vexp = (const double*)r.Vexp; u.X = (double*)Bw;
        u.col_stride = (int64_t)nb * ldw; u.tile_stride = nb; u.ld = ldw;
        u.group0 = 0; u.gstride = 1; u.k = k0; u.p = h->p; u.do_unmqr = 1;
        u.nsteps = q; u.nslc = (int)nslices; u.prog = (unsigned*)h->prog;
        u.vcol = p * h->vt; u.tcol = p * (int64_t)h->ib * nb; u.ecol = h->vt;
        u.w16 = h->w16 ? 1 : 0;
        CUDA_TRY(h, tqr::launch_update(nb, h->ib, 32, u, (int)(q * nslices), fwd, s));
        h->launches++;
        return TQR_OK;
    }
    for (int s_ = 0; s_ < q; ++s_) {
        const int k = fwd ? s_ : q - 1 - s_;
        Owner* O = h->local(h->owner_of[k]);
        const PanelRefs r = own_refs(h, *O, O->lidx[k]);
        CUDA_TRY(h, update(h, r, Bw, (int64_t)nb * ldw, nb, ldw, 0, 1, k, 32, (int)nslices, fwd, s, &h->launches));
    }
    return TQR_OK;
}

// Stage B (m x nrhs) into the zero-padded workspace (mp x nrhs rounded up to 32 columns).
static tqr_status stage_b(tqr_plan h, const void* B, int64_t ldb, int64_t nrhs, int64_t* nslices, cudaStream_t s) {
    const int64_t pad = (nrhs + 31) / 32 * 32;
    *nslices = pad / 32;
    const int64_t mp = (int64_t)h->p * h->nb;   // zero-padded rows m..mp-1 (Q = diag(Q_m, I))
    const size_t need = (size_t)mp * pad;
    const size_t es = h->es;
    if (need > h->bw_elems) {
        if (h->bw) cudaFree(h->bw);
        h->bw = nullptr;
        h->bw_elems = 0;
        CUDA_TRY(h, cudaMalloc(&h->bw, need * es));
        h->bw_elems = need;
    }
    CUDA_TRY(h, cudaMemsetAsync(h->bw, 0, need * es, s));
    CUDA_TRY(h, cudaMemcpy2DAsync(h->bw, mp * es, B, ldb * es, h->m * es, nrhs, cudaMemcpyDefault, s));
    return TQR_OK;
}

static tqr_status tqr_apply_qt_impl(tqr_plan h, char trans, void* B, int64_t ldb, int64_t nrhs) {
    NvtxRange nvtx_("tqr_apply_qt");
    if (!h) return TQR_ERR_ARG;
    if (h->poisoned) return fail(h, TQR_ERR_STATE, "plan poisoned by an earlier CUDA/NCCL failure");
    if (!h->factored) return fail(h, TQR_ERR_STATE, "apply_qt before a successful factor");
    if (!(trans == 'T' || trans == 't' || trans == 'N' || trans == 'n')) return fail(h, TQR_ERR_ARG, "trans must be 'T' or 'N'");
    if (nrhs < 0 || (nrhs > 0 && (!B || ldb < h->m))) return fail(h, TQR_ERR_ARG, "apply_qt: bad B/ldb/nrhs");
    if (nrhs == 0) return TQR_OK;
    if (h->rs) return rs_apply(h, trans, B, ldb, nrhs, false);
    if (needs_replica(h)) {
        tqr_status st = ensure_replica(h);
        if (!st) {
            st = tqr_apply_qt(h->rep, trans, B, ldb, nrhs);
            if (st) st = fail(h, st, "apply_qt (replica): %s", tqr_last_error(h->rep));
        }
        tqr_status sb = ipc_apply_barrier(h);
        return st ? st : sb;
    }
    int dev = 0;
    tqr_status st = single_device(h, &dev);
    if (st) return st;
    CUDA_TRY(h, cudaSetDevice(dev));
    cudaStream_t s = h->owners[0].s_upd;
    const size_t es = h->es;
    st = sync_entry(h, classify(B));
    if (st) return st;
    int64_t nsl = 0;
    st = stage_b(h, B, ldb, nrhs, &nsl, s);
    if (st) return st;
    const int64_t mp = (int64_t)h->p * h->nb;
    st = apply_device(h, trans, h->bw, mp, nsl, s);
    if (st) return st;
    CUDA_TRY(h, cudaMemcpy2DAsync(B, ldb * es, h->bw, mp * es, h->m * es, nrhs, cudaMemcpyDefault, s));
    CUDA_TRY(h, cudaStreamSynchronize(s));
    return TQR_OK;
}

static tqr_status tqr_solve_ls_impl(tqr_plan h, void* B, int64_t ldb, int64_t nrhs) {
    NvtxRange nvtx_("tqr_solve_ls");
    if (!h) return TQR_ERR_ARG;
    if (h->poisoned) return fail(h, TQR_ERR_STATE, "plan poisoned by an earlier CUDA/NCCL failure");
    if (!h->factored) return fail(h, TQR_ERR_STATE, "solve_ls before a successful factor");
    if (nrhs < 0 || (nrhs > 0 && (!B || ldb < h->m))) return fail(h, TQR_ERR_ARG, "solve_ls: bad B/ldb/nrhs");
    if (nrhs == 0) return TQR_OK;
    if (h->rs) return rs_apply(h, 'T', B, ldb, nrhs, true);
    if (needs_replica(h)) {
        tqr_status st = ensure_replica(h);
        if (!st) {
            st = tqr_solve_ls(h->rep, B, ldb, nrhs);
            if (st) st = fail(h, st, "solve_ls (replica): %s", tqr_last_error(h->rep));
        }
        tqr_status sb = ipc_apply_barrier(h);
        return st ? st : sb;
    }
    int dev = 0;
    tqr_status st = single_device(h, &dev);
    if (st) return st;
    CUDA_TRY(h, cudaSetDevice(dev));
    cudaStream_t s = h->owners[0].s_upd;
    const size_t es = h->es;
    st = sync_entry(h, classify(B));
    if (st) return st;
    int64_t nsl = 0;
    st = stage_b(h, B, ldb, nrhs, &nsl, s);
    if (st) return st;
    const int64_t mp = (int64_t)h->p * h->nb;
    st = apply_device(h, 'T', h->bw, mp, nsl, s);
    if (st) return st;
    // R X = (Q^T B)(0:n, :) by tile back substitution on the tile storage (trsm.cu): exact zero on
    // the diagonal first (LAPACK dtrtrs convention: TQR_ERR_SINGULAR, B unspecified)
    const int64_t n = h->n, nb = h->nb;
    const int64_t colsz = (int64_t)h->p * nb * nb;
    if (!h->dflag) CUDA_TRY(h, cudaMalloc(&h->dflag, sizeof(int64_t)));
    const unsigned long long big = ~0ull;
    CUDA_TRY(h, cudaMemcpyAsync(h->dflag, &big, sizeof(big), cudaMemcpyHostToDevice, s));
    for (auto& o : h->owners) {
        const int nc = (int)o.cols.size();
        auto* fz = reinterpret_cast<unsigned long long*>(h->dflag);
        if (h->f32()) CUDA_TRY(h, tqr::launch_diag_zero_tiles<float>((const float*)o.tiles, o.cols_dev, nc, colsz, (int)nb, n, fz, s));
        else CUDA_TRY(h, tqr::launch_diag_zero_tiles<double>((const double*)o.tiles, o.cols_dev, nc, colsz, (int)nb, n, fz, s));
        h->launches++;
    }
    unsigned long long first_zero = 0;
    CUDA_TRY(h, cudaMemcpyAsync(&first_zero, h->dflag, sizeof(first_zero), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(h, cudaStreamSynchronize(s));
    if (first_zero != big) return fail(h, TQR_ERR_SINGULAR, "R(%llu,%llu) == 0", first_zero, first_zero);
    for (int i = h->q - 1; i >= 0; --i) {
        Owner* O = h->local(h->owner_of[i]);
        const void* Rcol = h->at(O->tiles, (int64_t)O->lidx[i] * colsz);
        if (h->f32())
            CUDA_TRY(h, tqr::launch_trsm_step<float>((int)nb, (const float*)Rcol, i, (float*)h->bw, mp, n, (int)nsl, s));
        else
            CUDA_TRY(h, tqr::launch_trsm_step<double>((int)nb, (const double*)Rcol, i, (double*)h->bw, mp, n, (int)nsl, s));
        h->launches += (i > 0) ? 2 : 1;
    }
    CUDA_TRY(h, cudaMemcpy2DAsync(B, ldb * es, h->bw, mp * es, n * es, nrhs, cudaMemcpyDefault, s));
    CUDA_TRY(h, cudaStreamSynchronize(s));
    return TQR_OK;
}

// Every ABI entry point that can allocate on the host: no C++ exception crosses the boundary.
tqr_status tqr_create_ex(int64_t m, int64_t n, int32_t nb, int32_t ib, tqr_dtype dtype, int32_t ndev,
                         const int32_t* guide, int32_t guide_len, const tqr_options* opt, tqr_plan* out) {
    try {
        return tqr_create_ex_impl(m, n, nb, ib, dtype, ndev, guide, guide_len, opt, out);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_create_ex: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_create_ex: unexpected exception");
    }
}
tqr_status tqr_factor(tqr_plan h, void* A, int64_t lda) {
    try {
        return tqr_factor_impl(h, A, lda);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_factor: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_factor: unexpected exception");
    }
}
tqr_status tqr_load(tqr_plan h, const void* A, int64_t lda) {
    try {
        return tqr_load_impl(h, A, lda);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_load: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_load: unexpected exception");
    }
}
tqr_status tqr_factor_tiles(tqr_plan h) {
    try {
        return tqr_factor_tiles_impl(h);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_factor_tiles: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_factor_tiles: unexpected exception");
    }
}
tqr_status tqr_store_r(tqr_plan h, void* A, int64_t lda) {
    try {
        return tqr_store_r_impl(h, A, lda);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_store_r: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_store_r: unexpected exception");
    }
}
tqr_status tqr_apply_qt(tqr_plan h, char trans, void* B, int64_t ldb, int64_t nrhs) {
    try {
        return tqr_apply_qt_impl(h, trans, B, ldb, nrhs);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_apply_qt: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_apply_qt: unexpected exception");
    }
}
tqr_status tqr_solve_ls(tqr_plan h, void* B, int64_t ldb, int64_t nrhs) {
    try {
        return tqr_solve_ls_impl(h, B, ldb, nrhs);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_solve_ls: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_solve_ls: unexpected exception");
    }
}
tqr_status tqr_schedule(int64_t m, int64_t n, int32_t nb, int32_t ndev, const int32_t* guide, int32_t guide_len,
                        int32_t rank, int32_t* ops, int64_t cap, int64_t* count) {
    try {
        return tqr_schedule_impl(m, n, nb, ndev, guide, guide_len, rank, ops, cap, count);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_schedule: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_schedule: unexpected exception");
    }
}
tqr_status tqr_generate_guide(const int32_t* rates, int32_t ndev, int32_t* guide, int32_t cap, int32_t* len) {
    try {
        return tqr_generate_guide_impl(rates, ndev, guide, cap, len);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_generate_guide: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_generate_guide: unexpected exception");
    }
}
tqr_status tqr_ipc_connect(tqr_plan h, const void* all, int64_t len) {
    try {
        return tqr_ipc_connect_impl(h, all, len);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_ipc_connect: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_ipc_connect: unexpected exception");
    }
}
tqr_status tqr_ipc_handle(tqr_plan h, void* buf, int64_t cap, int64_t* len) {
    try {
        return tqr_ipc_handle_impl(h, buf, cap, len);
    } catch (const std::bad_alloc&) {
        return fail(nullptr, TQR_ERR_ALLOC, "tqr_ipc_handle: host allocation failed");
    } catch (...) {
        return fail(nullptr, TQR_ERR_ARG, "tqr_ipc_handle: unexpected exception");
    }
}

}  // extern "C"

// ------------------------------------------------------------------ NCCL loader
namespace tqr {
const NcclApi* nccl_api(const char** why) {
    static NcclApi api;
    static bool tried = false;
    static const char* reason = "not loaded";
    if (!tried) {
        tried = true;
        void* lib = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!lib) lib = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!lib) {
            reason = "dlopen(libnccl.so.2) failed";
        } else {
            bool ok = true;
            auto sym = [&](const char* n) { void* s = dlsym(lib, n); if (!s) ok = false; return s; };
            api.GetUniqueId = (decltype(api.GetUniqueId))sym("ncclGetUniqueId");
            api.CommInitRank = (decltype(api.CommInitRank))sym("ncclCommInitRank");
            api.CommDestroy = (decltype(api.CommDestroy))sym("ncclCommDestroy");
            api.CommGetAsyncError = (decltype(api.CommGetAsyncError))sym("ncclCommGetAsyncError");
            api.CommAbort = (decltype(api.CommAbort))sym("ncclCommAbort");
            api.Broadcast = (decltype(api.Broadcast))sym("ncclBroadcast");
            api.AllGather = (decltype(api.AllGather))sym("ncclAllGather");
            api.GroupStart = (decltype(api.GroupStart))sym("ncclGroupStart");
            api.GroupEnd = (decltype(api.GroupEnd))sym("ncclGroupEnd");
            api.GetErrorString = (decltype(api.GetErrorString))sym("ncclGetErrorString");
            api.ok = ok;
            if (!ok) reason = "libnccl.so.2 lacks a required symbol";
        }
    }
    if (!api.ok) { if (why) *why = reason; return nullptr; }
    return &api;
}
}  // namespace tqr
