// rgsqr_api.cu -- host driver and C-ABI (include/rgsqr.h) of the B200 RGSQR library.
//
// rgsqr_factor runs Algorithm 1 as a static, depth-first plan:
//   colnorm -> colscale -> scale/cast (section 3.5)
//   for each node of the recursion tree (left to right):
//     leaf   : panel (eq 8 + Alg 2, fp32)                               [+ allgather/stack]
//     inner  : K1 R12 = Q1^T A2 (tcgen05, split-K) -> reduce -> R, R12h   [+ allreduce]
//              K2 A2 -= Q1 R12 (tcgen05, fused fp32 RMW + 16-bit shadow)
//   unscale R (R <- R P^{-1}, exact)
// The plan (tensor maps, grid shapes, split factors) is built once per (shape, pointers,
// options) and captured into a CUDA graph, so a call is one graph launch.
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <map>
#include <mutex>
#include <climits>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <string>
#include <functional>
#include <vector>

#include "../../include/rgsqr.h"
#include "kernels.h"

// ------------------------------------------------------------------ NCCL (dlopen)
typedef struct ncclComm* ncclComm_t;
typedef struct {
    char internal[128];
} ncclUniqueId;
typedef enum { ncclSuccess = 0 } ncclResult_t;
typedef enum { ncclInt8 = 0, ncclFloat32 = 7, ncclFloat64 = 8 } ncclDataType_t;
typedef enum { ncclSum = 0 } ncclRedOp_t;

namespace {
struct NcclApi {
    void* lib = nullptr;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
};
NcclApi g_nccl;

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn g_encode = nullptr;

int64_t round_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }

int rgsqr_split(int64_t n) {  // reading #1: h = roundup(n/2, 32), clamped
    int64_t h = ((n / 2) + 31) / 32 * 32;
    if (h >= n) h = n / 2;
    if (h < 1) h = 1;
    return (int)h;
}

bool encode_map(CUtensorMap* map, const void* base, int64_t inner, int64_t outer, int64_t ld_elems, int box_inner,
                int box_outer, bool bf16) {
    if (!g_encode) return false;
    cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)outer};
    cuuint64_t strides[1] = {(cuuint64_t)(ld_elems * 2)};
    cuuint32_t box[2] = {(cuuint32_t)box_inner, (cuuint32_t)box_outer};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = g_encode(map, bf16 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2,
                          const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

// plain (unswizzled) 2-D map for the K2 TMA epilogue: fp32 (elem 4) or 16-bit (elem 2)
bool encode_plain(CUtensorMap* map, const void* base, int64_t inner, int64_t outer, int64_t ld_elems, int elem,
                  bool bf16, int box_inner, int box_outer) {
    if (!g_encode) return false;
    if ((reinterpret_cast<uintptr_t>(base) & 15) != 0 || ((ld_elems * elem) & 15) != 0) return false;
    cuuint64_t dims[2] = {(cuuint64_t)inner, (cuuint64_t)outer};
    cuuint64_t strides[1] = {(cuuint64_t)(ld_elems * elem)};
    cuuint32_t box[2] = {(cuuint32_t)box_inner, (cuuint32_t)box_outer};
    cuuint32_t estr[2] = {1, 1};
    const CUtensorMapDataType dt = elem == 4 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                   : bf16    ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16
                                             : CU_TENSOR_MAP_DATA_TYPE_FLOAT16;
    CUresult r = g_encode(map, dt, 2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                          CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

int pick_bn(int w) { return w <= 32 ? 32 : w <= 64 ? 64 : w <= 128 ? 128 : 256; }
// general GEMMs (lowrank): N > 256 takes 192-wide tiles when they waste fewer columns (N = 528:
// 3 x 192 = 576 instead of 3 x 256 = 768)
int pick_bn_general(int N) {
    if (N <= 256) return pick_bn(N);
    const int t256 = (N + 255) / 256 * 256, t192 = (N + 191) / 192 * 192;
    return t192 < t256 ? 192 : 256;
}

enum ProfClass { PC_UPDATE = 0, PC_PROJ = 1, PC_PANEL = 2, PC_SCALE = 3, PC_CGLS = 4, PC_OTHER = 5, PC_N = 6 };

}  // namespace

// ------------------------------------------------------------------ device buffers
// Workspace buffer of one handle.  A buffer is bound to its handle's stream and allocation epoch
// (rg_create): growing it bumps the epoch (plans / graphs embed addresses and are rebuilt) and
// zeroes the new memory in stream order on the handle's stream, then waits for it -- counters,
// flags and the leaf's grid-barrier word rely on zero-initialised workspace, and the handle's
// stream may be a non-blocking stream that the legacy-stream cudaMemset would not order against.
struct DevBuf {
    void* p = nullptr;
    size_t bytes = 0;
    int* epoch = nullptr;                 // owning handle's allocation epoch
    const cudaStream_t* stream = nullptr; // owning handle's stream
    bool ensure(size_t b) {
        if (b <= bytes) return true;
        if (epoch) ++*epoch;
        if (p) {
            if (stream) cudaStreamSynchronize(*stream);   // nothing in flight may still use it
            cudaFree(p);
        }
        p = nullptr;
        bytes = 0;
        if (cudaMalloc(&p, b) != cudaSuccess) {
            cudaGetLastError();
            p = nullptr;
            return false;
        }
        const cudaStream_t st = stream ? *stream : nullptr;
        if (cudaMemsetAsync(p, 0, b, st) != cudaSuccess || cudaStreamSynchronize(st) != cudaSuccess) {
            cudaFree(p);
            p = nullptr;
            return false;
        }
        bytes = b;
        return true;
    }
    void release() {
        if (p) cudaFree(p);
        p = nullptr;
        bytes = 0;
    }
    template <class T>
    T* as() const {
        return reinterpret_cast<T*>(p);
    }
};

struct Op {
    enum Kind { PANEL, PROJ, UPDATE, PAIR } kind;
    // PANEL: c0, w = columns.  PROJ/UPDATE: Q1 = [c0, c0+h), A2 = [c0+h, c0+h+w).
    // PAIR: the whole last recursion level [c0, c0+h+w) (h = 32) in one kernel.
    int c0, h, w;
    int bn = 0, tiles_i = 0, tiles_j = 0, splits = 0, kb_total = 0, kb_per_split = 0;
    CUtensorMap ma, mb, ma_lo, mb_lo;
    CUtensorMap mc;        // UPDATE: fp32 A2 for the TMA epilogue
    bool te = false;
    int h0 = 0;            // UPDATE: first output column whose 16-bit image a later K1 reads
    int a0 = -1;           // PROJ/UPDATE: first A2 column when not c0 + h (a column chunk of a level)
    int ref_w = 0;         // PROJ chunk: width of the whole level (its split-K decomposition is kept)
};
// first column of A2 (PROJ / UPDATE)
static inline int op_a2(const Op& o) { return o.a0 >= 0 ? o.a0 : o.c0 + o.h; }

// Host-pointer pipeline of rgsqr_factor (pinned host A/Q/R, one pass, one rank): A arrives in
// column chunks on a copy stream and each chunk is scaled (section 3.5) just before the first op
// that touches it; Q columns go back to the host as soon as their panel has run, because the
// recursion (Alg 1, eqs 4-5) only reads Q1 after its panel -- later levels write columns to the
// right of it.  Both PCIe directions then overlap the factorization instead of bracketing it.
struct HostPipe {
    float* hQ = nullptr;
    int64_t hldq = 0;
    float* hR = nullptr;
    int64_t hldr = 0;
    int chunk = 128;                  // H2D / scaling granularity (columns)
    int scaled = 0, copied = 0;       // columns scaled on the device / enqueued for D2H
    std::vector<cudaEvent_t>* in_ev = nullptr;   // H2D chunk k landed
    cudaStream_t cs_out = nullptr;
    cudaEvent_t ev = nullptr;         // main-stream progress marker for the D2H stream
};

struct Plan {
    // key
    int64_t m = 0, n = 0, lda = 0, ldq = 0, ldr = 0;
    const float* A = nullptr;
    float* Q = nullptr;
    float* R = nullptr;
    int nb = 0, bf16 = 0, split = 0, scale = 1, nranks = 1, rank = 0, panel = 0;
    int lazy = 0;   // > 0: column-lazy schedule with this chunk width (host-pointer pipeline)
    bool leaf = false;       // last level runs as leaf.cu kernels
    int epoch = -1;          // handle allocation epoch the plan was built against
    // derived
    int64_t ldh = 0, ldr12 = 0;
    std::vector<Op> ops;
    size_t p_floats = 0;
    long long launches = 0;  // kernels per pass (counted while enqueueing)
    cudaGraphExec_t exec = nullptr;
    HostPipe* pipe = nullptr;  // set for one eager enqueue of the host-pointer pipeline
};


// ------------------------------------------------------------------ in-process virtual ranks
// P handles on ONE device form a group; each rank's collective calls come from its own host
// thread (the API calls of the P ranks run concurrently, one thread per handle).  A collective
// is a host rendezvous: every rank records a "ready" event on its stream; the last to arrive
// makes its stream wait for all of them, reduces the P buffers in fixed rank order (0, 1, ..)
// into the group scratch with one kernel and copies the result to every rank's buffer (or, for
// an allgather, copies every rank's block into every rank's receive buffer), records "done",
// and wakes the others, which make their streams wait for "done".  Deterministic, no NCCL:
// it exists so that the row-sharded branches of the library can run and be
// checked on a single GPU (NCCL refuses two ranks on one device).
__global__ void vsum_kernel(const void* const* in, int P, size_t count, int f64, void* out) {
    const size_t stride = (size_t)gridDim.x * blockDim.x;
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < count; i += stride) {
        if (f64) {
            double s = reinterpret_cast<const double*>(in[0])[i];
            for (int r = 1; r < P; ++r) s += reinterpret_cast<const double*>(in[r])[i];
            reinterpret_cast<double*>(out)[i] = s;
        } else {
            float s = reinterpret_cast<const float*>(in[0])[i];
            for (int r = 1; r < P; ++r) s += reinterpret_cast<const float*>(in[r])[i];
            reinterpret_cast<float*>(out)[i] = s;
        }
    }
}

struct VGroup {
    int P = 0;
    int device = -1;
    std::mutex mu;
    std::condition_variable cv;
    int arrived = 0;
    unsigned long long gen = 0;
    int failed = 0;                      // a rank timed out or saw a mismatch: all later calls fail
    struct Slot {
        const void* send = nullptr;
        void* recv = nullptr;
        size_t count = 0;
        int kind = 0;                    // 0 allreduce (in place), 1 allgather
        int f64 = 0;
        cudaStream_t st = nullptr;
    };
    std::vector<Slot> slots;
    std::vector<cudaEvent_t> ready;
    cudaEvent_t done = nullptr;
    void* scratch = nullptr;             // reduction result
    size_t scratch_bytes = 0;
    void** dptrs = nullptr;              // device array of the P input pointers
    int attached = 0;
};

int vgroup_collective(VGroup* g, int rank, VGroup::Slot slot) {
    using namespace std::chrono;
    std::unique_lock<std::mutex> lk(g->mu);
    if (g->failed) return RG_NCCL_ERROR;
    if (cudaEventRecord(g->ready[rank], slot.st) != cudaSuccess) return RG_CUDA_ERROR;
    g->slots[rank] = slot;
    const unsigned long long my = g->gen;
    if (++g->arrived == g->P) {
        int rc = RG_OK;
        for (int r = 0; r < g->P; ++r)
            if (g->slots[r].count != slot.count || g->slots[r].kind != slot.kind || g->slots[r].f64 != slot.f64)
                rc = RG_NCCL_ERROR;   // ranks disagree on the collective: a library bug
        cudaStream_t st = slot.st;
        const size_t esz = slot.f64 ? 8 : 4, bytes = slot.count * esz;
        for (int r = 0; r < g->P && rc == RG_OK; ++r)
            if (cudaStreamWaitEvent(st, g->ready[r], 0) != cudaSuccess) rc = RG_CUDA_ERROR;
        if (rc == RG_OK && slot.kind == 0 && bytes > 0) {
            if (bytes > g->scratch_bytes) {
                cudaStreamSynchronize(st);
                if (g->scratch) cudaFree(g->scratch);
                g->scratch = nullptr;
                g->scratch_bytes = 0;
                if (cudaMalloc(&g->scratch, bytes) != cudaSuccess) rc = RG_ALLOC;
                else g->scratch_bytes = bytes;
            }
            std::vector<const void*> in((size_t)g->P);
            for (int r = 0; r < g->P; ++r) in[r] = g->slots[r].recv;
            if (rc == RG_OK &&
                cudaMemcpyAsync(g->dptrs, in.data(), sizeof(void*) * g->P, cudaMemcpyHostToDevice, st) != cudaSuccess)
                rc = RG_CUDA_ERROR;
            if (rc == RG_OK) {
                // (the host array `in` must outlive the async copy: synchronise before it goes away)
                const int blocks = (int)std::min<size_t>(1024, (slot.count + 255) / 256);
                vsum_kernel<<<blocks, 256, 0, st>>>(const_cast<const void* const*>(g->dptrs), g->P, slot.count,
                                                    slot.f64, g->scratch);
                ++rg::g_launches;
                if (cudaGetLastError() != cudaSuccess || cudaStreamSynchronize(st) != cudaSuccess) rc = RG_CUDA_ERROR;
            }
            for (int r = 0; r < g->P && rc == RG_OK; ++r)
                if (cudaMemcpyAsync(g->slots[r].recv, g->scratch, bytes, cudaMemcpyDeviceToDevice, st) != cudaSuccess)
                    rc = RG_CUDA_ERROR;
        } else if (rc == RG_OK && slot.kind == 1 && bytes > 0) {
            for (int r = 0; r < g->P && rc == RG_OK; ++r)
                for (int q = 0; q < g->P && rc == RG_OK; ++q) {
                    char* dst = reinterpret_cast<char*>(g->slots[r].recv) + (size_t)q * bytes;
                    if (dst == g->slots[q].send) continue;
                    if (cudaMemcpyAsync(dst, g->slots[q].send, bytes, cudaMemcpyDeviceToDevice, st) != cudaSuccess)
                        rc = RG_CUDA_ERROR;
                }
        }
        if (rc == RG_OK && cudaEventRecord(g->done, st) != cudaSuccess) rc = RG_CUDA_ERROR;
        if (rc) g->failed = 1;
        g->arrived = 0;
        ++g->gen;
        g->cv.notify_all();
        return rc;
    }
    if (!g->cv.wait_for(lk, seconds(120), [&] { return g->gen != my; })) {
        g->failed = 1;   // a peer rank never arrived (it returned early with an error)
        g->cv.notify_all();
        return RG_NCCL_ERROR;
    }
    if (g->failed) return RG_NCCL_ERROR;
    return cudaStreamWaitEvent(slot.st, g->done, 0) == cudaSuccess ? RG_OK : RG_CUDA_ERROR;
}

struct rg_handle_s {
    int device = 0;
    cudaStream_t stream = nullptr;
    cudaStream_t capture_stream = nullptr;  // private stream used only to capture plans into graphs
    cudaStream_t cs_in = nullptr, cs_out = nullptr;   // host-pointer pipeline copy streams (lazy)
    std::vector<cudaEvent_t> pipe_ev;               // [0] progress, [1] start, [2] end, [3..] H2D chunks
    ncclComm_t comm = nullptr;       // NCCL communicator (row-sharded mode)
    bool own_comm = false;           // created by rg_comm_init (destroyed with the handle)
    VGroup* vgroup = nullptr;        // in-process virtual ranks (rg_set_vcomm)
    bool dist() const { return nranks > 1 && (comm || vgroup); }
    int rank = 0, nranks = 1;
    int64_t last_info = -1;
    // workspace
    DevBuf cq_ws, cq_flags;                         // CholQR2 panel workspace (flags: fail, counters)
    DevBuf leaf_bar;                                // grid-barrier word of the leaf kernel
    DevBuf qh, ql, P, r12h, r12l, r12f, partial, norm2, scale, status, pws, pcnt, rgather, rstackq;
    DevBuf stageA, stageQ, stageR, stageB, stageX;  // host-pointer staging
    DevBuf cg;                                      // CGLS vectors
    DevBuf lsQ, lsR, rinv, probeG, probeW;          // ls_solve_refined / orthogonalize workspace
    DevBuf lrA16, lrB16, lrB16l, lrY, lrZ, lrQ16, lrQ16l, lrR, lrW, lrV, lrUb, lrVb, lrSig, lrOm, lrScale, lrFlags;
    cudaGraphExec_t cgls_exec = nullptr;            // captured block of CGLS iterations
    const void* cgls_key[4] = {nullptr, nullptr, nullptr, nullptr};
    int64_t cgls_key_mn[3] = {0, 0, 0};
    int cgls_solver = -1;                           // solver the captured block was built for
    bool cgls_one_pass = false;                     // this solve's CGLS product (reading #24)
    bool cgls_graph_one_pass = false;               // product the captured block was built with
    DevBuf aux;                                     // misc (orthogonalize / lowrank)
    DevBuf tallws;                                  // tall CholQR pass (tall.cu)
    DevBuf vscratch;                                // virtual-rank collectives (rank 0 of a group)
    int alloc_epoch = 0;                            // bumped whenever a workspace buffer moves
    std::vector<DevBuf*> bufs() {
        return {&qh, &ql, &P, &r12h, &r12l, &r12f, &partial, &norm2, &scale, &status, &pws, &pcnt,
                &rgather, &rstackq, &stageA, &stageQ, &stageR, &stageB, &stageX, &cg, &aux, &lsQ, &lsR, &rinv,
                &probeG, &probeW, &cq_ws, &cq_flags, &leaf_bar, &lrA16, &lrB16, &lrB16l, &lrY, &lrZ, &lrQ16,
                &lrQ16l, &lrR, &lrW, &lrV, &lrUb, &lrVb, &lrSig, &lrOm, &lrScale, &lrFlags, &vscratch, &tallws};
    }
    void bind_bufs() {
        for (DevBuf* b : bufs()) {
            b->epoch = &alloc_epoch;
            b->stream = &stream;
        }
    }
    int* status_host = nullptr;                     // pinned
    long long last_launches = 0;                    // kernels launched by the last API call
    long long call_g0 = 0;                          // rg::g_launches at the start of the call
    long long replayed = 0;                         // kernels in CUDA-graph replays of this call
    std::vector<std::unique_ptr<Plan>> plans;      // LRU, most recent first
    // profiling
    bool prof = false;
    double prof_ms[PC_N] = {0};
    int64_t prof_launches[PC_N] = {0};
    double prof_flops[PC_N] = {0};
    double prof_bytes[PC_N] = {0};
    std::vector<std::pair<cudaEvent_t, cudaEvent_t>> ev_pool;
    struct PendingEv {
        int cls;
        cudaEvent_t a, b;
        double flops, bytes;
        int tag;   // op width tag for the RGSQR_PROF_OPS per-op trace (kind * 100000 + w)
    };
    std::vector<PendingEv> pending;
    size_t ev_next = 0;
};

namespace {

#define RG_CUDA(x)                                                                   \
    do {                                                                             \
        cudaError_t _e = (x);                                                        \
        if (_e != cudaSuccess) {                                                     \
            fprintf(stderr, "[rgsqr] CUDA error %s at %s:%d: %s\n", cudaGetErrorName(_e), __FILE__, __LINE__, \
                    cudaGetErrorString(_e));                                         \
            return RG_CUDA_ERROR;                                                    \
        }                                                                            \
    } while (0)

// profiling brackets ------------------------------------------------------------
struct ProfScope {
    rg_handle h;
    int cls;
    double flops, bytes;
    int tag;
    cudaEvent_t b = nullptr, e = nullptr;
    ProfScope(rg_handle h_, int cls_, double flops_ = 0, double bytes_ = 0, int tag_ = 0)
        : h(h_), cls(cls_), flops(flops_), bytes(bytes_), tag(tag_) {
        if (!h->prof) return;
        if (h->ev_next >= h->ev_pool.size()) {
            cudaEvent_t x, y;
            cudaEventCreate(&x);
            cudaEventCreate(&y);
            h->ev_pool.push_back({x, y});
        }
        b = h->ev_pool[h->ev_next].first;
        e = h->ev_pool[h->ev_next].second;
        h->ev_next++;
        cudaEventRecord(b, h->stream);
    }
    ~ProfScope() {
        if (!h->prof) return;
        cudaEventRecord(e, h->stream);
        h->pending.push_back({cls, b, e, flops, bytes, tag});
    }
};

void prof_collect(rg_handle h) {
    if (!h->prof || h->pending.empty()) return;
    cudaStreamSynchronize(h->stream);
    static const bool trace = getenv("RGSQR_PROF_OPS") != nullptr;
    for (auto& p : h->pending) {
        float ms = 0;
        cudaEventElapsedTime(&ms, p.a, p.b);
        if (trace)
            fprintf(stderr, "[rgsqr op] cls %d w %d us %.2f TF %.1f GB/s %.0f\n", p.cls, p.tag, ms * 1e3,
                    p.flops / (ms * 1e-3) / 1e12, p.bytes / (ms * 1e-3) / 1e9);
        h->prof_ms[p.cls] += ms;
        h->prof_launches[p.cls] += 1;
        h->prof_flops[p.cls] += p.flops;
        h->prof_bytes[p.cls] += p.bytes;
    }
    h->pending.clear();
    h->ev_next = 0;
}

bool ensure_encode() {
    if (g_encode) return true;
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess || !fn)
        return false;
    g_encode = reinterpret_cast<EncodeTiledFn>(fn);
    return true;
}

enum PtrSide { SIDE_DEVICE, SIDE_HOST };
// page-locked (cudaHostAlloc / cudaHostRegister) host memory: copies to and from it are async DMA
bool is_pinned(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return a.type == cudaMemoryTypeHost;
}

PtrSide ptr_side(const void* p) {
    cudaPointerAttributes a;
    if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
        cudaGetLastError();
        return SIDE_HOST;
    }
    return (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) ? SIDE_DEVICE : SIDE_HOST;
}

// ------------------------------------------------------------------ plan construction
void build_ops(std::vector<Op>& ops, int c0, int ncols, int nb, bool pair, bool leaf) {
    if (pair && (ncols > nb || leaf) && ncols <= 2 * nb) {
        Op o{};
        o.kind = Op::PAIR;
        o.c0 = c0;
        o.h = rgsqr_split(ncols);
        o.w = ncols - o.h;
        ops.push_back(o);
        return;
    }
    if (ncols <= nb) {
        Op o{};
        o.kind = Op::PANEL;
        o.c0 = c0;
        o.w = ncols;
        ops.push_back(o);
        return;
    }
    const int h = rgsqr_split(ncols), w = ncols - h;
    build_ops(ops, c0, h, nb, pair, leaf);
    Op p{};
    p.kind = Op::PROJ;
    p.c0 = c0;
    p.h = h;
    p.w = w;
    ops.push_back(p);
    Op u = p;
    u.kind = Op::UPDATE;
    ops.push_back(u);
    build_ops(ops, c0 + h, w, nb, pair, leaf);
}

// PROJ op oi (and the UPDATE after it) of the level just above a leaf, run as the leaf's prologue
bool folded_into_leaf(const Plan& pl, size_t oi) {
static const bool no_fold64 = getenv("RGSQR_NO_FOLD64") != nullptr;
const auto& ops = pl.ops;
const Op& o = ops[oi];
return pl.leaf && !no_fold64 && rg::leaf_prologue_fits(pl.m) && o.kind == Op::PROJ && o.h <= 64 && o.w <= 64 &&
       oi + 2 < ops.size() && ops[oi + 1].kind == Op::UPDATE && ops[oi + 1].c0 == o.c0 &&
       ops[oi + 2].kind == Op::PAIR && ops[oi + 2].c0 == o.c0 + o.h && ops[oi + 2].h + ops[oi + 2].w == o.w &&
       o.a0 < 0;
}

// Column-lazy schedule of the recursion for the host-pointer pipeline: the K1 / K2 pair of every
// level wider than C is applied to its A2 in C-column chunks, each chunk just before the first op
// that touches those columns (and after every earlier level's chunks on them), instead of all at
// once.  Per column the updates are the same, in the same order (Alg 1's recursion); what changes is
// only when they run -- so the factorization can follow the column-chunked H2D of A instead of
// waiting for the whole right half before the top level's K1 (the e2e bound of the eager order:
// H2D(A) + D2H(right half of Q)).
void lazy_schedule(std::vector<Op>& ops, int C) {
    struct Pend {
        Op proj;
        std::vector<char> done;
    };
    std::vector<Pend> pend;
    std::vector<Op> out;
    out.reserve(ops.size() * 2);
    std::function<void(int, int, size_t)> flush = [&](int x0, int x1, size_t upto) {
        for (size_t r = 0; r < upto && r < pend.size(); ++r) {
            Pend& p = pend[r];
            const int a = op_a2(p.proj);
            for (size_t k = 0; k < p.done.size(); ++k) {
                const int s0 = a + (int)k * C, s1 = std::min(a + p.proj.w, s0 + C);
                if (p.done[k] || s1 <= x0 || s0 >= x1) continue;
                flush(s0, s1, r);   // earlier levels first on these columns
                p.done[k] = 1;
                Op pr = p.proj;
                pr.a0 = s0;
                pr.w = s1 - s0;
                pr.ref_w = p.proj.w;
                out.push_back(pr);
                Op up = pr;
                up.kind = Op::UPDATE;
                up.ref_w = 0;
                out.push_back(up);
            }
        }
    };
    for (size_t i = 0; i < ops.size(); ++i) {
        const Op& o = ops[i];
        if (o.kind == Op::PROJ && o.w > C) {
            Pend p;
            p.proj = o;
            p.done.assign((size_t)((o.w + C - 1) / C), 0);
            pend.push_back(p);
            ++i;   // its UPDATE
            continue;
        }
        int x0, x1;
        if (o.kind == Op::PANEL) x0 = o.c0, x1 = o.c0 + o.w;
        else if (o.kind == Op::PAIR) x0 = o.c0, x1 = o.c0 + o.h + o.w;
        else x0 = op_a2(o), x1 = op_a2(o) + o.w;
        flush(x0, x1, pend.size());
        out.push_back(o);
    }
    flush(0, INT_MAX, pend.size());
    ops.swap(out);
}

int make_plan(rg_handle h, Plan& pl) {
    if (!ensure_encode()) return RG_CUDA_ERROR;
    const int64_t m = pl.m;
    const int n = (int)pl.n;
    pl.ldh = round_up(std::max<int64_t>(m, 8), 8);
    pl.ops.clear();
    // The last recursion level (two 32-column panels + K1 + K2 of a <= 64-column block) runs as
    // one kernel when the rows per SM fit in shared memory: by default the leaf kernel (leaf.cu,
    // the paper's structure with rows resident on chip); opt-in RGSQR_WIDE=1 the 64-column
    // CholQR2 kernel (same Q, R in exact arithmetic).
    const bool wide = getenv("RGSQR_WIDE") != nullptr;
    // Figure 7 ablation: RGSQR_NO_TC=1 runs K1 / K2 as fp32 SIMT GEMMs and the panels
    // without the leaf's 16-bit tensor-core paths (single GPU only; development switch)
    const bool no_tc = getenv("RGSQR_NO_TC") != nullptr && !(pl.nranks > 1 && h->dist());
    // (split-precision passes keep the tensor-core K1/K2 at the last level: the leaf kernel's
    // mma.sync K1/K2 are single 16-bit products)
    const bool pair = !no_tc && pl.panel == 0 && pl.nb == 32 && !(pl.nranks > 1 && h->dist()) &&
                      (wide ? rg::cholqr_fused_fits(m, 64) : (rg::leaf_fits(m) && !pl.split));
    pl.leaf = pair && !wide;
    build_ops(pl.ops, 0, n, pl.nb, pair, pl.leaf);
    if (pl.lazy > 0) lazy_schedule(pl.ops, pl.lazy);
    // 16-bit images written by K2 that nothing reads: a column's image is read only as A2 of a
    // later K1 before the leaf / panel that factors the column (those read fp32 and write the
    // image of Q).  In leaf mode that drops the image for the first 128 columns of every K2
    // output (the w = 128 level writes none).
    {
        std::vector<int> last((size_t)n, -1);   // UPDATE op that last wrote the column's image
        std::vector<int> need(pl.ops.size(), INT_MAX);
        for (size_t i = 0; i < pl.ops.size(); ++i) {
            const Op& o = pl.ops[i];
            if (o.kind == Op::PROJ && !folded_into_leaf(pl, i)) {   // (a folded prologue reads fp32)
                for (int c = op_a2(o); c < op_a2(o) + o.w; ++c)
                    if (last[c] >= 0) need[last[c]] = std::min(need[last[c]], c);
            } else if (o.kind == Op::UPDATE) {
                for (int c = op_a2(o); c < op_a2(o) + o.w; ++c) last[c] = (int)i;
            } else {
                const int c1 = o.kind == Op::PAIR ? o.c0 + o.h + o.w : o.c0 + o.w;
                for (int c = o.c0; c < c1; ++c) last[c] = -2;
            }
        }
        for (size_t i = 0; i < pl.ops.size(); ++i)
            if (pl.ops[i].kind == Op::UPDATE) {
                Op& o = pl.ops[i];
                o.h0 = need[i] == INT_MAX ? o.w : std::max(0, need[i] - op_a2(o));
            }
    }
    int max_h = 0, max_w = 0;
    size_t pmax = 0;
    for (auto& o : pl.ops)
        if (o.kind == Op::PROJ || o.kind == Op::UPDATE) {
            max_h = std::max(max_h, o.h);
            max_w = std::max(max_w, o.w);
        }
    pl.ldr12 = round_up(std::max(max_h, 8), 8);
    const uint16_t* qh = h->qh.as<uint16_t>();
    const uint16_t* ql = h->ql.as<uint16_t>();
    const uint16_t* r12h = h->r12h.as<uint16_t>();
    const uint16_t* r12l = h->r12l.as<uint16_t>();
    const bool bf = pl.bf16 != 0;
    for (auto& o : pl.ops) {
        if (o.kind == Op::PANEL || o.kind == Op::PAIR) continue;
        const uint16_t* q1 = qh + (int64_t)o.c0 * pl.ldh;
        const uint16_t* a2 = qh + (int64_t)op_a2(o) * pl.ldh;
        const uint16_t* q1l = pl.split ? ql + (int64_t)o.c0 * pl.ldh : q1;
        const uint16_t* a2l = pl.split ? ql + (int64_t)op_a2(o) * pl.ldh : a2;
        o.bn = pick_bn(o.w);
        if (o.kind == Op::UPDATE && getenv("RGSQR_K2_BN")) o.bn = std::min(o.bn, atoi(getenv("RGSQR_K2_BN")));
        if (o.kind == Op::PROJ) {
            o.tiles_i = (o.h + 127) / 128;
            o.tiles_j = (o.w + o.bn - 1) / o.bn;
            o.kb_total = (int)((m + 63) / 64);
            // a column chunk of a level keeps the whole level's split-K decomposition (the same
            // partial sums in the same order: bit-identical R12 / Q to the unchunked plan)
            const int sw = o.ref_w > 0 ? o.ref_w : o.w, sbn = pick_bn(sw);
            const int tiles = o.tiles_i * ((sw + sbn - 1) / sbn);
            int splits = 1;
            if (tiles >= 32) {
                // balance whole waves of 148 persistent CTAs against split-K partial traffic
                double best = -1.0;
                for (int s = 1; s <= std::min(32, std::max(1, o.kb_total / 8)); ++s) {
                    const double units = (double)tiles * s;
                    const double eff = units / 148.0 / std::ceil(units / 148.0) - 0.01 * s;
                    if (eff > best + 1e-9) {
                        best = eff;
                        splits = s;
                    }
                }
            } else {
                // small outputs are bandwidth/latency bound: spread the m rows over ~one wave
                splits = std::max(1, std::min(148 / tiles, o.kb_total / 8));
            }
            o.kb_per_split = (o.kb_total + splits - 1) / splits;
            o.splits = (o.kb_total + o.kb_per_split - 1) / o.kb_per_split;
            pmax = std::max(pmax, (size_t)o.splits * o.tiles_j * o.bn * o.tiles_i * 128);
            bool ok = encode_map(&o.ma, q1, m, o.h, pl.ldh, 64, 128, bf) &&
                      encode_map(&o.mb, a2, m, o.w, pl.ldh, 64, o.bn, bf) &&
                      encode_map(&o.ma_lo, q1l, m, o.h, pl.ldh, 64, 128, bf) &&
                      encode_map(&o.mb_lo, a2l, m, o.w, pl.ldh, 64, o.bn, bf);
            if (!ok) return RG_CUDA_ERROR;
        } else {
            o.te = !pl.split && encode_plain(&o.mc, pl.Q + (int64_t)op_a2(o) * pl.ldq, m, o.w, pl.ldq, 4, bf, 128, 32);
            bool ok = encode_map(&o.ma, q1, m, o.h, pl.ldh, 64, 64, bf) &&
                      encode_map(&o.mb, r12h, o.h, o.w, pl.ldr12, 64, o.bn, bf) &&
                      encode_map(&o.ma_lo, q1l, m, o.h, pl.ldh, 64, 64, bf) &&
                      // non-split: the lo slot carries the half-width B box of the cluster-pair K2
                      encode_map(&o.mb_lo, pl.split ? r12l : r12h, o.h, o.w, pl.ldr12, 64, pl.split ? o.bn : std::max(8, o.bn / 2), bf);
            if (!ok) return RG_CUDA_ERROR;
        }
    }
    if (no_tc)
        for (auto& o : pl.ops)
            if (o.kind == Op::PROJ) pmax = std::max(pmax, rg::sgemm_tn_work_floats(m, o.h, o.w));
    pl.p_floats = pmax;
    (void)max_w;
    return RG_OK;
}

// grow every workspace buffer the plan needs; returns false on allocation failure
bool ensure_workspace(rg_handle h, int64_t m, int64_t n, int split) {
    const int64_t ldh = round_up(std::max<int64_t>(m, 8), 8);
    const size_t qh_bytes = (size_t)ldh * n * 2;
    // projection partials: bounded by splits * padded tiles; computed generously here
    const int64_t hmax = n / 2 + 32, wmax = n / 2 + 32;
    bool ok = h->qh.ensure(qh_bytes) && (!split || h->ql.ensure(qh_bytes)) &&
              h->r12h.ensure((size_t)round_up(hmax, 8) * wmax * 2 + 4096) &&
              (!split || h->r12l.ensure((size_t)round_up(hmax, 8) * wmax * 2 + 4096)) &&
              h->r12f.ensure((size_t)hmax * wmax * 4 + 4096) &&
              h->partial.ensure(rg::colnorm_partial_doubles(m, (int)n) * 8 + 64) && h->norm2.ensure(n * 8 + 64) &&
              h->scale.ensure(n * 4 + 64) && h->status.ensure(64) &&
              h->pws.ensure(rg::panel_ws_floats(m) * 4 + 4096) && h->pcnt.ensure(rg::panel_counters(m) * 4 + 64) &&
              h->rgather.ensure((size_t)64 * 32 * 32 * 4) && h->rstackq.ensure((size_t)64 * 32 * 32 * 4) &&
              h->cq_ws.ensure(std::max(rg::cholqr_ws_doubles(m), rg::leaf_ws_doubles()) * 8 + 256) &&
              h->leaf_bar.ensure(4096) &&
              h->cq_flags.ensure((rg::cholqr_counter_ints(m) + 8) * 4);
    return ok;
}

// in-place sum over the ranks (no-op on one rank)
int nccl_allreduce(rg_handle h, void* buf, size_t count, ncclDataType_t t) {
    if (!h->dist()) return RG_OK;
    if (h->vgroup) {
        VGroup::Slot sl;
        sl.send = buf;
        sl.recv = buf;
        sl.count = count;
        sl.kind = 0;
        sl.f64 = t == ncclFloat64;
        sl.st = h->stream;
        return vgroup_collective(h->vgroup, h->rank, sl);
    }
    if (g_nccl.AllReduce(buf, buf, count, t, ncclSum, h->comm, h->stream) != ncclSuccess) return RG_NCCL_ERROR;
    return RG_OK;
}

// recv[r * count ..] = rank r's send (count elements each, fp32)
int coll_allgather_f32(rg_handle h, const float* send, float* recv, size_t count) {
    if (h->vgroup) {
        VGroup::Slot sl;
        sl.send = send;
        sl.recv = recv;
        sl.count = count;
        sl.kind = 1;
        sl.f64 = 0;
        sl.st = h->stream;
        return vgroup_collective(h->vgroup, h->rank, sl);
    }
    if (g_nccl.AllGather(send, recv, count, ncclFloat32, h->comm, h->stream) != ncclSuccess) return RG_NCCL_ERROR;
    return RG_OK;
}

// enqueue one RGSQR pass on h->stream (no sync).  A -> Q (may alias), R (ldr).
int enqueue_rgsqr_impl(rg_handle h, Plan& pl);
int enqueue_rgsqr(rg_handle h, Plan& pl) {
    const long long before = rg::g_launches;
    int rc = enqueue_rgsqr_impl(h, pl);
    pl.launches = rg::g_launches - before;
    return rc;
}
int enqueue_rgsqr_impl(rg_handle h, Plan& pl) {
    cudaStream_t st = h->stream;
    const int64_t m = pl.m;
    const int n = (int)pl.n;
    uint16_t* qh = h->qh.as<uint16_t>();
    uint16_t* ql = pl.split ? h->ql.as<uint16_t>() : nullptr;
    int* status = h->status.as<int>();
    const bool dist = pl.nranks > 1 && h->dist();
    const bool no_tc = getenv("RGSQR_NO_TC") != nullptr && !dist;
    HostPipe* pp = pl.pipe;
    // section 3.5 on columns [c, c + nc): norms, power-of-two scales, scaled fp32 + 16-bit images
    auto scale_cols = [&](int c, int nc) -> int {
        RG_CUDA(rg::launch_colnorm(pl.A + (int64_t)c * pl.lda, pl.lda, m, nc, h->partial.as<double>(),
                                   h->norm2.as<double>() + c, st));
        RG_CUDA(rg::launch_colscale(h->norm2.as<double>() + c, nc, pl.scale, h->scale.as<float>() + c, status, c, st));
        RG_CUDA(rg::launch_scale_cast(pl.A + (int64_t)c * pl.lda, pl.lda, pl.Q + (int64_t)c * pl.ldq, pl.ldq,
                                      qh + (int64_t)c * pl.ldh, ql ? ql + (int64_t)c * pl.ldh : nullptr, pl.ldh, m, nc,
                                      h->scale.as<float>() + c, pl.bf16, st));
        return RG_OK;
    };
    // pipeline: scale the columns [pp->scaled, cend) rounded up to whole chunks, each after its H2D
    auto pipe_need = [&](int cend) -> int {
        while (pp && pp->scaled < cend) {
            const int c = pp->scaled, nc = std::min(pp->chunk, n - c);
            RG_CUDA(cudaStreamWaitEvent(st, (*pp->in_ev)[c / pp->chunk], 0));
            int rc = scale_cols(c, nc);
            if (rc) return rc;
            pp->scaled += nc;
        }
        return RG_OK;
    };
    // pipeline: Q columns [0, cend) are final; send the new ones home in >= 256-column pieces
    auto pipe_done = [&](int cend, bool flush) -> int {
        if (!pp || cend - pp->copied <= 0 || (!flush && cend - pp->copied < 256)) return RG_OK;
        // R(:, j) is final once column j's panel has run too (eq 6: R12 blocks of column j come
        // from K1s of levels where j lies in A2, all enqueued before that panel)
        RG_CUDA(rg::launch_unscale_r(pl.R, pl.ldr, n, pl.scale > 0 ? h->scale.as<float>() : nullptr, st, pp->copied,
                                     cend - pp->copied));
        RG_CUDA(cudaEventRecord(pp->ev, st));
        RG_CUDA(cudaStreamWaitEvent(pp->cs_out, pp->ev, 0));
        RG_CUDA(cudaMemcpy2DAsync(pp->hQ + (int64_t)pp->copied * pp->hldq, pp->hldq * 4,
                                  pl.Q + (int64_t)pp->copied * pl.ldq, pl.ldq * 4, m * 4, cend - pp->copied,
                                  cudaMemcpyDeviceToHost, pp->cs_out));
        RG_CUDA(cudaMemcpy2DAsync(pp->hR + (int64_t)pp->copied * pp->hldr, pp->hldr * 4,
                                  pl.R + (int64_t)pp->copied * pl.ldr, pl.ldr * 4, n * 4, cend - pp->copied,
                                  cudaMemcpyDeviceToHost, pp->cs_out));
        pp->copied = cend;
        return RG_OK;
    };
    int panel_end = 0;   // columns left of this have had their panel enqueued
    if (pp) {
        RG_CUDA(cudaMemset2DAsync(pl.R, pl.ldr * sizeof(float), 0, n * sizeof(float), n, st));
    } else if (pl.scale < 0) {
        // reorthogonalisation pass (reading #32): the input is the previous pass's Q, in place and
        // unscaled -- no norm pass, no fp32 copy; only the 16-bit images are written
        ProfScope _s(h, PC_SCALE, 0, (double)m * n * (pl.split ? 8 : 6));
        RG_CUDA(rg::launch_scale_cast(pl.A, pl.lda, nullptr, 0, qh, ql, pl.ldh, m, n, nullptr, pl.bf16, st));
        RG_CUDA(cudaMemset2DAsync(pl.R, pl.ldr * sizeof(float), 0, n * sizeof(float), n, st));
    } else {
        ProfScope _s(h, PC_SCALE, 0, (double)m * n * (pl.split ? 16 : 14));
        RG_CUDA(rg::launch_colnorm(pl.A, pl.lda, m, n, h->partial.as<double>(), h->norm2.as<double>(), st));
        if (dist) {
            int rc = nccl_allreduce(h, h->norm2.p, n, ncclFloat64);
            if (rc) return rc;
        }
        RG_CUDA(rg::launch_colscale(h->norm2.as<double>(), n, pl.scale, h->scale.as<float>(), status, 0, st));
        RG_CUDA(rg::launch_scale_cast(pl.A, pl.lda, pl.Q, pl.ldq, qh, ql, pl.ldh, m, n, h->scale.as<float>(), pl.bf16,
                                      st));
        RG_CUDA(cudaMemset2DAsync(pl.R, pl.ldr * sizeof(float), 0, n * sizeof(float), n, st));
    }
    const Op* pending_update = nullptr;   // leaf-level K2 folded into the next panel's load
    const Op* pending_pro = nullptr;      // K1 + K2 of the level above a leaf, folded into it
    for (size_t oi = 0; oi < pl.ops.size(); ++oi) {
        const Op& o = pl.ops[oi];
        if (pp) {
            int rc = pipe_done(panel_end, false);
            if (!rc) rc = pipe_need(o.kind == Op::PANEL ? o.c0 + o.w : o.kind == Op::PAIR ? o.c0 + o.h + o.w : op_a2(o) + o.w);
            if (rc) return rc;
        }
        if (folded_into_leaf(pl, oi)) {
            pending_pro = &o;
            ++oi;   // the UPDATE too
            continue;
        }
        if (o.kind == Op::UPDATE && !dist && pl.panel == 0 && o.h <= 64 && oi + 1 < pl.ops.size() &&
            pl.ops[oi + 1].kind == Op::PANEL && pl.ops[oi + 1].c0 == o.c0 + o.h && pl.ops[oi + 1].w == o.w && o.a0 < 0 &&
            rg::cholqr_fused_fits(m, 32) && getenv("RGSQR_NO_FOLD") == nullptr) {
            pending_update = &o;
            continue;
        }
        if (o.kind == Op::PAIR) {
            panel_end = o.c0 + o.h + o.w;
            // two panels + R12 = Q1^T A2 + A2 -= Q1 R12 of a (h + w)-column block; algorithmic bytes:
            // read the block (fp32), write Q (fp32) + shadow(s)
            const double wt = o.h + o.w;
            ProfScope _s(h, PC_PANEL, 2.0 * m * (o.h * o.h + o.w * o.w) + 4.0 * m * o.h * o.w,
                         (double)m * wt * (pl.split ? 12 : 10), pending_pro ? 1 : 0);   // tag 1: folded prologue
            int* cq_fail = h->cq_flags.as<int>();
            rg::CholqrLaunch c{};
            c.P = pl.Q + (int64_t)o.c0 * pl.ldq;
            c.ldp = pl.ldq;
            c.Q = pl.Q + (int64_t)o.c0 * pl.ldq;
            c.ldq = pl.ldq;
            c.Qh = qh + (int64_t)o.c0 * pl.ldh;
            c.Ql = ql ? ql + (int64_t)o.c0 * pl.ldh : nullptr;
            c.ldh = pl.ldh;
            c.m = m;
            c.nc = o.h + o.w;
            c.ws = h->cq_ws.as<double>();
            c.counter = cq_fail + 4;
            c.fail = cq_fail;
            c.R = pl.R + o.c0 + (int64_t)o.c0 * pl.ldr;
            c.ldr = pl.ldr;
            c.bf16 = pl.bf16;
            c.status = status;
            c.col0 = o.c0;
            if (getenv("RGSQR_WIDE") != nullptr) {
                RG_CUDA(rg::launch_panel_pair(c, st));
            } else {
                rg::LeafLaunch L{};
                L.Q = c.Q;
                L.ldq = c.ldq;
                L.Qh = c.Qh;
                L.Ql = c.Ql;
                L.ldh = c.ldh;
                L.m = m;
                L.nc = c.nc;
                L.R = c.R;
                L.ldr = c.ldr;
                L.ws = h->cq_ws.as<double>();
                L.bar = h->leaf_bar.as<unsigned>();
                L.status = status;
                L.col0 = o.c0;
                L.bf16 = pl.bf16;
                if (pending_pro) {
                    L.pq = qh + (int64_t)pending_pro->c0 * pl.ldh;
                    L.ph = pending_pro->h;
                    pending_pro = nullptr;
                }
                RG_CUDA(rg::launch_leaf(L, st));
            }
            continue;
        }
        if (o.kind == Op::PANEL) {
            panel_end = o.c0 + o.w;
            // algorithmic bytes: read the panel (fp32), write Q (fp32) + 16-bit shadow (+ lo shadow)
            ProfScope _s(h, PC_PANEL, 2.0 * m * o.w * o.w, (double)m * o.w * (pl.split ? 12 : 10), o.w);
            rg::PanelLaunch p{};
            p.Q = pl.Q + (int64_t)o.c0 * pl.ldq;
            p.ldq = pl.ldq;
            p.Qh = qh + (int64_t)o.c0 * pl.ldh;
            p.Ql = ql ? ql + (int64_t)o.c0 * pl.ldh : nullptr;
            p.ldh = pl.ldh;
            p.m = m;
            p.nc = o.w;
            p.ws = h->pws.as<float>();
            p.counters = h->pcnt.as<int>();
            p.bf16 = pl.bf16;
            p.col0 = o.c0;
            p.status = status;
            float* Rdiag = pl.R + o.c0 + (int64_t)o.c0 * pl.ldr;
            int* cq_fail = h->cq_flags.as<int>();
            int* cq_counters = cq_fail + 4;
            if (pl.panel == 0) {
                // CholQR2 (fp64 Gram); the MGS/TSQR kernels below run only if a pivot failed
                rg::CholqrLaunch c{};
                c.P = p.Q;
                c.ldp = pl.ldq;
                c.Q = p.Q;
                c.ldq = pl.ldq;
                c.Qh = p.Qh;
                c.Ql = p.Ql;
                c.ldh = pl.ldh;
                c.m = m;
                c.nc = o.w;
                c.ws = h->cq_ws.as<double>();
                c.counter = cq_counters;
                c.fail = cq_fail;
                c.R = Rdiag;
                c.ldr = pl.ldr;
                c.bf16 = pl.bf16;
                if (dist) {
                    c.allreduce_g = [](double* G, void* ctx) {
                        return nccl_allreduce(reinterpret_cast<rg_handle>(ctx), G, 1024, ncclFloat64);
                    };
                    c.ctx = h;
                }
                p.guard = cq_fail;
                c.status = status;
                c.col0 = o.c0;
                if (pending_update) {
                    const Op& u = *pending_update;
                    c.uq = pl.Q + (int64_t)u.c0 * pl.ldq;
                    c.uq_ld = pl.ldq;
                    c.ur = pl.R + u.c0 + (int64_t)(u.c0 + u.h) * pl.ldr;
                    c.ur_ld = pl.ldr;
                    c.uh = u.h;
                    pending_update = nullptr;
                }
                bool handled = false;
                RG_CUDA(rg::launch_panel_cholqr(c, &handled, st));
                if (handled) continue;   // shifted CholQR3 fallback inside the fused kernel
            }
            if (!dist) {
                p.R = Rdiag;
                p.ldr = pl.ldr;
                p.distributed = 0;
                RG_CUDA(rg::launch_panel(p, st));
            } else {
                // local TSQR -> gather the P local R's -> redundant stack MGS -> apply own block
                float* rg_all = h->rgather.as<float>();
                p.R = rg_all + (int64_t)h->rank * o.w * o.w;
                p.ldr = o.w;
                p.distributed = 1;
                RG_CUDA(rg::launch_panel(p, st));
                int rc = coll_allgather_f32(h, p.R, rg_all, (size_t)o.w * o.w);
                if (rc) return rc;
                float* qb = h->rstackq.as<float>();
                RG_CUDA(rg::launch_panel_stack(rg_all, h->nranks, o.w, Rdiag, pl.ldr, qb, status, o.c0, p.guard, st));
                RG_CUDA(rg::launch_panel_apply(p, qb + (int64_t)h->rank * 32 * 32, st));
            }
        } else if (o.kind == Op::PROJ && no_tc) {
            ProfScope _s(h, PC_PROJ, 2.0 * m * o.h * o.w, (double)m * (o.h + o.w) * 4, o.w);
            RG_CUDA(rg::launch_sgemm_proj(pl.Q + (int64_t)o.c0 * pl.ldq, pl.Q + (int64_t)op_a2(o) * pl.ldq, pl.ldq, m,
                                          o.h, o.w, pl.R + o.c0 + (int64_t)op_a2(o) * pl.ldr, pl.ldr,
                                          h->P.as<float>(), st));
        } else if (o.kind == Op::UPDATE && no_tc) {
            ProfScope _s(h, PC_UPDATE, 2.0 * m * o.h * o.w, (double)m * o.h * 4 + (double)m * o.w * 8, o.w);
            RG_CUDA(rg::launch_sgemm_update(pl.Q + (int64_t)o.c0 * pl.ldq, pl.R + o.c0 + (int64_t)op_a2(o) * pl.ldr,
                                            pl.ldr, pl.Q + (int64_t)op_a2(o) * pl.ldq, pl.ldq, m, o.h, o.w, st));
        } else if (o.kind == Op::PROJ) {
            ProfScope _s(h, PC_PROJ, 2.0 * m * o.h * o.w * (pl.split ? 3 : 1),
                             (double)m * (o.h + o.w) * (pl.split ? 4 : 2), o.w);
            float* P = h->P.as<float>();
            const int64_t ldp = (int64_t)o.tiles_i * 128;
            const int64_t pstride = ldp * o.tiles_j * o.bn;
            RG_CUDA(rg::launch_proj_gemm(o.bn, pl.split != 0, o.tiles_i, o.tiles_j, o.splits, o.ma, o.mb, o.ma_lo,
                                         o.mb_lo, P, ldp, pstride, o.kb_total, o.kb_per_split, pl.bf16, st));
            float* Rblk = pl.R + o.c0 + (int64_t)op_a2(o) * pl.ldr;
            uint16_t* r12l = pl.split ? h->r12l.as<uint16_t>() : nullptr;
            if (!dist) {
                RG_CUDA(rg::launch_proj_reduce(P, ldp, pstride, o.splits, o.h, o.w, Rblk, pl.ldr, nullptr, 0,
                                               h->r12h.as<uint16_t>(), r12l, pl.ldr12, pl.bf16, st));
            } else {
                float* rf = h->r12f.as<float>();
                RG_CUDA(rg::launch_proj_reduce(P, ldp, pstride, o.splits, o.h, o.w, nullptr, 0, rf, o.h, nullptr,
                                               nullptr, 0, pl.bf16, st));
                int rc = nccl_allreduce(h, rf, (size_t)o.h * o.w, ncclFloat32);
                if (rc) return rc;
                RG_CUDA(rg::launch_proj_finish(rf, o.h, o.h, o.w, Rblk, pl.ldr, h->r12h.as<uint16_t>(), r12l, pl.ldr12,
                                               pl.bf16, st));
            }
        } else {
            ProfScope _s(h, PC_UPDATE, 2.0 * m * o.h * o.w * (pl.split ? 3 : 1),
                             (double)m * o.h * (pl.split ? 4 : 2) + (double)m * o.w * (pl.split ? 12 : 10), o.w);
            float* C = pl.Q + (int64_t)op_a2(o) * pl.ldq;
            uint16_t* Ch = qh + (int64_t)op_a2(o) * pl.ldh;
            uint16_t* Cl = ql ? ql + (int64_t)op_a2(o) * pl.ldh : nullptr;
            RG_CUDA(rg::launch_update_gemm(o.bn, pl.split != 0, m, o.w, o.h, o.ma, o.mb, o.ma_lo, o.mb_lo, C, pl.ldq, Ch,
                                           Cl, pl.ldh, pl.bf16, st, 0, o.te ? &o.mc : nullptr, o.h0));
        }
    }
    if (pp) {
        int rc = pipe_need(n);
        if (!rc) rc = pipe_done(n, true);
        return rc;   // R unscaled and sent home piecewise
    }
    {
        ProfScope _s(h, PC_OTHER);
        RG_CUDA(rg::launch_unscale_r(pl.R, pl.ldr, n, pl.scale > 0 ? h->scale.as<float>() : nullptr, st));
    }
    return RG_OK;
}

void begin_call(rg_handle h) {
    h->call_g0 = rg::g_launches;
    h->replayed = 0;
    h->last_launches = 0;
}
void end_call(rg_handle h) { h->last_launches = (rg::g_launches - h->call_g0) + h->replayed; }

int reset_status(rg_handle h) {
    static const int init[4] = {INT_MAX, INT_MAX, 0, 0};
    RG_CUDA(cudaMemcpyAsync(h->status.p, init, sizeof(init), cudaMemcpyHostToDevice, h->stream));
    return RG_OK;
}

int check_status(rg_handle h) {
    RG_CUDA(cudaMemcpyAsync(h->status_host, h->status.p, 4 * sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    RG_CUDA(cudaStreamSynchronize(h->stream));
    h->last_info = -1;
    if (h->status_host[1] != INT_MAX) {
        h->last_info = h->status_host[1];
        return RG_NONFINITE;
    }
    if (h->status_host[0] != INT_MAX) {
        h->last_info = h->status_host[0];
        return RG_BREAKDOWN;
    }
    return RG_OK;
}

// run one RGSQR pass (device pointers), with an LRU cache of plans + CUDA graph replay.
// local = true forces the single-GPU path even in row-sharded mode (used for the small
// replicated factorizations of lowrank_approx).
int run_rgsqr(rg_handle h, int64_t m, int64_t n, const float* A, int64_t lda, float* Q, int64_t ldq, float* R,
              int64_t ldr, const rg_opts& o, int split, bool local = false, HostPipe* pipe = nullptr) {
    if (!ensure_workspace(h, m, n, split)) return RG_ALLOC;
    if (o.scale < 0 && (A != Q || lda != ldq || pipe)) return RG_CUDA_ERROR;   // reortho form: in place only
    const int nb = (o.nb <= 0 || o.nb > 32) ? 32 : o.nb;
    const int nranks = local ? 1 : h->nranks;
    static const int pipe_chunk = getenv("RGSQR_PIPE_LAZY") ? atoi(getenv("RGSQR_PIPE_LAZY")) : 256;
    const int lazy = pipe ? pipe_chunk : 0;
    Plan* pl = nullptr;
    for (size_t i = 0; i < h->plans.size(); ++i) {
        Plan* c = h->plans[i].get();
        if (c->m == m && c->n == n && c->lda == lda && c->ldq == ldq && c->ldr == ldr && c->A == A && c->Q == Q &&
            c->R == R && c->nb == nb && c->bf16 == o.precision && c->split == split && c->scale == o.scale &&
            c->nranks == nranks && c->rank == h->rank && c->panel == o.panel && c->lazy == lazy) {
            if (c->epoch != h->alloc_epoch) {   // a workspace buffer moved: rebuild this plan
                if (c->exec) cudaGraphExecDestroy(c->exec);
                h->plans.erase(h->plans.begin() + i);
                break;
            }
            pl = c;
            std::rotate(h->plans.begin(), h->plans.begin() + i, h->plans.begin() + i + 1);   // most recent first
            break;
        }
    }
    if (!pl) {
        std::unique_ptr<Plan> np(new Plan());
        np->m = m; np->n = n; np->lda = lda; np->ldq = ldq; np->ldr = ldr;
        np->A = A; np->Q = Q; np->R = R;
        np->nb = nb; np->bf16 = o.precision; np->split = split; np->scale = o.scale;
        np->nranks = nranks; np->rank = h->rank; np->panel = o.panel; np->lazy = lazy;
        int rc = make_plan(h, *np);
        if (rc) return rc;
        if (!h->P.ensure(np->p_floats * 4 + 4096)) return RG_ALLOC;
        np->epoch = h->alloc_epoch;
        // invalidate older plans if P just moved (their graphs captured the old pointer)
        for (auto& c : h->plans)
            if (c->epoch != h->alloc_epoch && c->exec) {
                cudaGraphExecDestroy(c->exec);
                c->exec = nullptr;
            }
        h->plans.insert(h->plans.begin(), std::move(np));
        while (h->plans.size() > 8) {
            if (h->plans.back()->exec) cudaGraphExecDestroy(h->plans.back()->exec);
            h->plans.pop_back();
        }
        pl = h->plans.front().get();
    }
    int rc = reset_status(h);
    if (rc) return rc;
    if (pipe) {   // eager: the copy-stream waits sit between the plan's kernels
        const long long graph_launches = pl->launches;
        pl->pipe = pipe;
        rc = enqueue_rgsqr(h, *pl);
        pl->pipe = nullptr;
        pl->launches = graph_launches;
        return rc;
    }
    const bool use_graph = !h->prof && !h->vgroup && getenv("RGSQR_NO_GRAPH") == nullptr;
    if (!use_graph) return enqueue_rgsqr(h, *pl);
    if (!pl->exec) {
        // capture on the private stream (the user's may be the legacy stream, which cannot
        // capture); the instantiated graph is then launched on the user's stream
        cudaGraph_t g;
        cudaStream_t user = h->stream;
        h->stream = h->capture_stream;
        RG_CUDA(cudaStreamBeginCapture(h->stream, cudaStreamCaptureModeThreadLocal));
        const long long cap0 = rg::g_launches;
        rc = enqueue_rgsqr(h, *pl);
        rg::g_launches = cap0;   // captured, not launched: the replay below is counted instead
        cudaError_t ce = cudaStreamEndCapture(h->stream, &g);
        h->stream = user;
        if (rc) {
            if (ce == cudaSuccess) cudaGraphDestroy(g);
            return rc;
        }
        RG_CUDA(ce);
        cudaError_t ie = cudaGraphInstantiate(&pl->exec, g, 0);
        cudaGraphDestroy(g);
        RG_CUDA(ie);
    }
    RG_CUDA(cudaGraphLaunch(pl->exec, h->stream));
    h->replayed += pl->launches;
    return RG_OK;
}

// R <- R2 R (both upper triangular n x n), via a scratch copy
int trmm_into(rg_handle h, const float* R2, int64_t ld2, float* R, int64_t ldr, int n) {
    if (!h->aux.ensure((size_t)n * n * 4 + 256)) return RG_ALLOC;
    float* Rt = h->aux.as<float>();
    RG_CUDA(rg::launch_trmm_upper(R2, ld2, R, ldr, Rt, n, n, h->stream));
    RG_CUDA(cudaMemcpy2DAsync(R, ldr * 4, Rt, (size_t)n * 4, (size_t)n * 4, n, cudaMemcpyDeviceToDevice, h->stream));
    return RG_OK;
}

// Hutchinson estimate of ||I - Q^T Q||_F with 8 fixed Philox probes (fp64), synchronous.
int orth_estimate(rg_handle h, const float* Q, int64_t ldq, int64_t m, int n, double* est) {
    const size_t pw = rg::probe_work_doubles(m, n, 8) + (size_t)n * 8 + 16;
    if (!h->probeG.ensure((size_t)n * 8 * 8 + 64) || !h->probeW.ensure(pw * 8)) return RG_ALLOC;
    double* G = h->probeG.as<double>();
    double* Z = h->probeW.as<double>();
    double* W = Z + (size_t)n * 8;
    double* out = W + rg::probe_work_doubles(m, n, 8);
    RG_CUDA(rg::launch_gaussian_philox((int64_t)n * 8, 0x5EEDCAFEULL, G, nullptr, h->stream));
    RG_CUDA(rg::launch_orth_probe_z(Q, ldq, m, n, G, W, Z, h->stream));
    int rc = nccl_allreduce(h, Z, (size_t)n * 8, ncclFloat64);
    if (rc) return rc;
    RG_CUDA(rg::launch_orth_probe_finish(Z, n, G, out, h->stream));
    double v = 0;
    RG_CUDA(cudaMemcpyAsync(&v, out, sizeof(double), cudaMemcpyDeviceToHost, h->stream));
    RG_CUDA(cudaStreamSynchronize(h->stream));
    *est = sqrt(v);
    return RG_OK;
}

// One tall CholQR pass (tall.cu, reading #33) in place on X (m_local x n, n <= 256): Gram on the
// tensor cores (+ allreduce of the n x n Gram when row-sharded), Cholesky / inverse / kappa test,
// X <- X R^-1; Rp (n x n, ld ldrp) = R.  *ok = false (X untouched) when the Cholesky broke down or
// kappa_F of the equilibrated R exceeds 32 n: the caller falls back to an RGSQR pass.
// first: the pass over the user's A (bf16 split, no column scaling needed); otherwise a
// reorthogonalisation pass over unit columns (fp16 split at scale 2^14).
bool tall_wanted(rg_handle h, int64_t m_local, int64_t n, const float* X, int64_t ldx) {
    const char* e = getenv("RGSQR_TALL");
    if (e && e[0] == '0') return false;
    (void)X;
    (void)ldx;
    if (n < 1 || n > 256) return false;
    if (e && e[0] == '1') return true;
    return !rg::leaf_fits(m_local) && m_local >= 4 * n;
}
// Gram of X (tall.cu) into the workspace's G, allreduced when row-sharded.  first: the pass over
// the user's A (bf16 split, no column scaling needed); otherwise unit columns (fp16 split, 2^14).
constexpr float kTallSig = 16384.0f;
int tall_gram(rg_handle h, int64_t m, int n, const float* X, int64_t ldx, bool first) {
    if (!h->tallws.ensure(rg::tall_ws_bytes())) return RG_ALLOC;
    double* G = rg::tall_gram_buffer(h->tallws.p);
    CUtensorMap tm;
    const bool tma = ensure_encode() && encode_plain(&tm, X, m, n, ldx, 4, false, 64, 128);
    RG_CUDA(rg::launch_tall_gram(X, ldx, m, n, first ? 1.0f : kTallSig, first ? 1 : 0, h->tallws.p, G, h->stream,
                                 tma ? &tm : nullptr));
    if (getenv("RGSQR_TALL_DEBUG")) {   // tensor-core diagonal against the fp64 column sums
        std::vector<double> dg((size_t)n), dt((size_t)n);
        RG_CUDA(cudaStreamSynchronize(h->stream));
        RG_CUDA(cudaMemcpy(dt.data(), rg::tall_dbg(h->tallws.p), n * 8, cudaMemcpyDeviceToHost));
        RG_CUDA(cudaMemcpy2D(dg.data(), 8, G, (size_t)(n + 1) * 8, 8, n, cudaMemcpyDeviceToHost));
        double mx = 0, sq = 0;
        for (int i = 0; i < n; ++i) {
            const double r = dt[i] / dg[i] - 1.0;
            mx = std::max(mx, std::fabs(r));
            sq += r * r;
        }
        fprintf(stderr, "[tall] gram m=%lld first=%d: tensor-core diagonal vs fp64 norms: max rel %.3g rms %.3g\n",
                (long long)m, (int)first, mx, std::sqrt(sq / n));
    }
    return nccl_allreduce(h, G, (size_t)n * n, ncclFloat64);
}
// ||I - X^T X||_F from the Gram just formed by tall_gram(first = false) (synchronous)
int tall_orth(rg_handle h, int n, double* est) {
    double* G = rg::tall_gram_buffer(h->tallws.p);
    double* out = rg::tall_kout(h->tallws.p) + 2;
    RG_CUDA(rg::launch_tall_orth(G, n, (double)kTallSig, out, h->stream));
    RG_CUDA(cudaMemcpyAsync(est, out, sizeof(double), cudaMemcpyDeviceToHost, h->stream));
    RG_CUDA(cudaStreamSynchronize(h->stream));
    return RG_OK;
}
// Cholesky / inverse / kappa test of the Gram from tall_gram, then X <- X R^-1 in place and
// Rp (n x n, ld ldrp) = R.  *ok = false (X untouched) when the Cholesky broke down or kappa_F of the
// equilibrated R exceeds 32 n: the caller falls back to an RGSQR pass.
int tall_chol_apply(rg_handle h, int64_t m, int n, float* X, int64_t ldx, float* Rp, int64_t ldrp, bool first,
                    bool* ok) {
    void* ws = h->tallws.p;
    // the Gram's scale (bf16 split at 1 on the first pass: the column norms are unknown before it);
    // the apply always splits in fp16 at 2^14: X D^-1 has unit columns once the Gram gave D
    const float sig_g = first ? 1.0f : kTallSig;
    const int apply_bf16 = getenv("RGSQR_TALL_APPLY_BF16") ? (first ? 1 : 0) : 0;
    RG_CUDA(rg::launch_tall_chol_apply(X, ldx, m, n, rg::tall_gram_buffer(ws), (double)sig_g,
                                       apply_bf16 ? 1.0f : kTallSig, apply_bf16, 32.0 * n, Rp, ldrp, ws, h->stream));
    int flag = 0;
    RG_CUDA(cudaMemcpyAsync(&flag, rg::tall_flag(ws), sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    RG_CUDA(cudaStreamSynchronize(h->stream));
    *ok = flag == 0;
    if (getenv("RGSQR_TALL_DEBUG")) {
        double k[2] = {0, 0};
        RG_CUDA(cudaMemcpy(k, rg::tall_kout(ws), sizeof(k), cudaMemcpyDeviceToHost));
        fprintf(stderr, "[tall] m=%lld n=%d first=%d flag=%d kappa_F=%.4g (limit %.4g) pivot=%g\n", (long long)m, n,
                (int)first, flag, k[0], 32.0 * n, k[1]);
    }
    return RG_OK;
}

// run RGSQR + `extra` reorthogonalisation passes (16-bit; split precision with opts.split) for the
// least-squares preconditioner; Q (ldq) and R (ldr) outputs
int factor_with_reortho(rg_handle h, int64_t m, int64_t n, const float* A, int64_t lda, float* Q, int64_t ldq, float* R,
                        int64_t ldr, const rg_opts& o, int extra) {
    int rc = run_rgsqr(h, m, n, A, lda, Q, ldq, R, ldr, o, o.split);
    for (int p = 0; p < extra && rc == RG_OK; ++p) {
        if (o.sync) {
            rc = check_status(h);
            if (rc) return rc;
        }
        if (!h->lsR.ensure((size_t)n * n * 4 + 256)) return RG_ALLOC;
        float* R2 = h->lsR.as<float>();
        // reading #8: for the CGLS preconditioner a plain 16-bit reortho pass suffices (kappa(A R^-1)
        // ~ 1.8 either way, SURVEY [EMU]); split precision only when the caller asks (opts.split)
        rg_opts o2 = o;
        o2.scale = -1;   // in place, unscaled (reading #32)
        rc = run_rgsqr(h, m, n, Q, ldq, Q, ldq, R2, n, o2, o.split);
        if (rc) return rc;
        rc = trmm_into(h, R2, n, R, ldr, (int)n);
    }
    return rc;
}

// CGLS iterations (Alg 3 corrected, readings #5-#7) on device vectors; R^{-1} explicit (fp64).
int enqueue_cgls_iters(rg_handle h, const float* A, int64_t lda, int64_t m, int n, int iters, double* base) {
    cudaStream_t st = h->stream;
    double* sc = base;
    double* Rinv = h->rinv.as<double>();
    double* x = sc + 16;
    double* p = x + n;
    double* s = p + n;
    double* t = s + n;
    double* sv = t + n;
    double* r = sv + n;
    double* q = r + m;
    double* work = q + m;
    double* sqp = work + std::max({rg::gemv_n_work_doubles(m, n), rg::gemv_t_work_doubles(m, n),
                                   rg::gemv_nt_work_doubles(n) + (size_t)n});
    const double* done = sc + 6;
    if (h->cgls_one_pass) {
        // one pass over A per iteration: q = A t and w = A^T q together; A^T r by recurrence
        double* w = work + rg::gemv_nt_work_doubles(n);
        for (int k = 0; k < iters; ++k) {
            ProfScope _s(h, PC_CGLS, 4.0 * m * n, 4.0 * m * n);
            RG_CUDA(rg::launch_trmv(Rinv, n, p, t, 0, done, st));                 // t = R \ p
            RG_CUDA(rg::launch_gemv_nt(A, lda, m, n, t, q, w, work, sc, st));    // q = A t, w = A^T q, delta
            int rc = nccl_allreduce(h, sc + 1, 1, ncclFloat64);
            if (rc) return rc;
            rc = nccl_allreduce(h, w, n, ncclFloat64);
            if (rc) return rc;
            RG_CUDA(rg::launch_cgls_xr(x, t, r, q, m, n, sc, st));                 // lines 13-15 (alpha)
            RG_CUDA(rg::launch_cgls_sv(sv, w, n, sc, st));                         // A^T r -= alpha A^T q
            RG_CUDA(rg::launch_trmv(Rinv, n, sv, s, 1, done, st));                // line 16: s = R^-T A^T r
            RG_CUDA(rg::launch_cgls_p(s, p, n, sc, 0, st));                        // lines 17-21
        }
        return RG_OK;
    }
    for (int k = 0; k < iters; ++k) {
        ProfScope _s(h, PC_CGLS, 4.0 * m * n, 8.0 * m * n);
        RG_CUDA(rg::launch_trmv(Rinv, n, p, t, 0, done, st));                 // t = R \ p
        // line 11: q = A t; line 12: delta = |q|^2 (partials from the split sums, fixed order)
        RG_CUDA(rg::launch_gemv_n(A, lda, m, n, t, q, work, done, st, sc, 1, sqp));
        int rc = nccl_allreduce(h, sc + 1, 1, ncclFloat64);
        if (rc) return rc;
        RG_CUDA(rg::launch_cgls_xr(x, t, r, q, m, n, sc, st));                 // lines 13-15
        RG_CUDA(rg::launch_gemv_t(A, lda, m, n, r, sv, work, done, st));        // A^T r
        rc = nccl_allreduce(h, sv, n, ncclFloat64);
        if (rc) return rc;
        RG_CUDA(rg::launch_trmv(Rinv, n, sv, s, 1, done, st));                // line 16: s = R^-T A^T r
        RG_CUDA(rg::launch_cgls_p(s, p, n, sc, 0, st));                        // lines 17-21
    }
    return RG_OK;
}


// LSQR iterations (NEXT-4) on the same buffers: base = sc[16] | y v w t sv p (n each) | u q (m each) |
// work.  Two passes over A per iteration like CGLS; dist: |u|^2 and A^T u allreduced.
int enqueue_lsqr_iters(rg_handle h, const float* A, int64_t lda, int64_t m, int n, int iters, double* base) {
    cudaStream_t st = h->stream;
    double* sc = base;
    double* y = sc + 16;
    double* v = y + n;
    double* w = v + n;
    double* t = w + n;
    double* sv = t + n;
    double* p = sv + n;
    double* u = p + n;
    double* q = u + m;
    double* work = q + m;
    double* wnt = work + rg::gemv_nt_work_doubles(n);   // one-pass: A^T q
    double* sqp = work + std::max({rg::gemv_n_work_doubles(m, n), rg::gemv_t_work_doubles(m, n),
                                   rg::gemv_nt_work_doubles(n) + (size_t)n});
    double* Rinv = h->rinv.as<double>();
    const double* done = sc + 6;
    const bool one = h->cgls_one_pass;
    for (int k = 0; k < iters; ++k) {
        ProfScope _s(h, PC_CGLS, 4.0 * m * n, (one ? 4.0 : 8.0) * m * n);
        RG_CUDA(rg::launch_trmv(Rinv, n, v, t, 0, done, st));                       // t = R^-1 v
        if (one)   // q = A t and A^T q in one sweep of A (reading #24)
            RG_CUDA(rg::launch_gemv_nt(A, lda, m, n, t, q, wnt, work, sc, st));
        else
            RG_CUDA(rg::launch_gemv_n(A, lda, m, n, t, q, work, done, st));        // q = A t = M v
        RG_CUDA(rg::launch_lsqr_u(u, q, m, sc, sqp, st));                          // u = q - alpha u, |u|^2
        int rc = nccl_allreduce(h, sc + 1, 1, ncclFloat64);
        if (rc) return rc;
        if (one) {
            rc = nccl_allreduce(h, wnt, n, ncclFloat64);
            if (rc) return rc;
            RG_CUDA(rg::launch_lsqr_sv(sv, wnt, n, sc, st));                       // A^T u by recurrence
        } else {
            RG_CUDA(rg::launch_gemv_t(A, lda, m, n, u, sv, work, done, st));       // A^T u
            rc = nccl_allreduce(h, sv, n, ncclFloat64);
            if (rc) return rc;
        }
        RG_CUDA(rg::launch_trmv(Rinv, n, sv, p, 1, done, st));                     // p = R^-T A^T u
        RG_CUDA(rg::launch_lsqr_step(p, v, w, y, n, sc, 0, st));                   // v, alpha, Givens, y, w
    }
    return RG_OK;
}

// ------------------------------------------------------------------ general GEMMs (lowrank)
// C (m x N fp32, ldc) = A (m x K, MN-major 16-bit, lda16) * B (K x N, K-major 16-bit, ldb16);
// split: A_lo / B_lo images give ~fp32 accuracy (reading #9).
int gemm_nn(rg_handle h, int64_t m, int N, int K, const uint16_t* Ah, const uint16_t* Al, int64_t lda16,
            const uint16_t* Bh, const uint16_t* Bl, int64_t ldb16, float* C, int64_t ldc, int bf16) {
    const int bn = pick_bn_general(N);
    CUtensorMap ma, mb, mal, mbl;
    const bool split = Al && Bl;
    if (!encode_map(&ma, Ah, m, K, lda16, 64, 64, bf16) || !encode_map(&mb, Bh, K, N, ldb16, 64, bn, bf16) ||
        !encode_map(&mal, split ? Al : Ah, m, K, lda16, 64, 64, bf16) ||
        !encode_map(&mbl, split ? Bl : Bh, K, N, ldb16, 64, bn, bf16))
        return RG_CUDA_ERROR;
    RG_CUDA(rg::launch_update_gemm(bn, split, m, N, K, ma, mb, mal, mbl, C, ldc, nullptr, nullptr, 0, bf16, h->stream,
                                   1));
    return RG_OK;
}

// O (M x N fp32, ldo) = A^T B with A (K x M, K-major 16-bit, lda16) and B (K x N, lda16
// layout ldb16): split-K over the K = m rows + deterministic reduction (K1 kernels).
int gemm_tn(rg_handle h, int64_t K, int M, int N, const uint16_t* Ah, int64_t lda16, const uint16_t* Bh,
            int64_t ldb16, float* O, int64_t ldo, int bf16) {
    const int bn = pick_bn_general(N);
    CUtensorMap ma, mb;
    if (!encode_map(&ma, Ah, K, M, lda16, 64, 128, bf16) || !encode_map(&mb, Bh, K, N, ldb16, 64, bn, bf16))
        return RG_CUDA_ERROR;
    const int tiles_i = (M + 127) / 128, tiles_j = (N + bn - 1) / bn;
    const int kb_total = (int)((K + 63) / 64);
    const int tiles = tiles_i * tiles_j;
    int splits = tiles >= 148 ? 1 : std::max(1, std::min(148 / tiles, kb_total / 8));
    const int kps = (kb_total + splits - 1) / splits;
    splits = (kb_total + kps - 1) / kps;
    const int64_t ldp = (int64_t)tiles_i * 128;
    const int64_t pstride = ldp * tiles_j * bn;
    if (!h->P.ensure((size_t)splits * pstride * 4 + 4096)) return RG_ALLOC;
    float* P = h->P.as<float>();
    // A (M = the rows of the output: e.g. lowrank's 32768 columns of A, 2 GB) is the operand too large
    // for L2: units enumerate the N tiles fastest so each A tile is read from HBM once
    RG_CUDA(rg::launch_proj_gemm(bn, false, tiles_i, tiles_j, splits, ma, mb, ma, mb, P, ldp, pstride, kb_total, kps,
                                 bf16, h->stream, 1));
    RG_CUDA(rg::launch_proj_reduce(P, ldp, pstride, splits, M, N, nullptr, 0, O, ldo, nullptr, nullptr, 0, bf16,
                                   h->stream));
    return RG_OK;
}
}  // namespace

namespace rg {
thread_local long long g_launches = 0;
bool pdl_enabled() {   // opt-in: measured slower than plain graph edges for this kernel mix
    static const bool on = getenv("RGSQR_PDL") != nullptr;
    return on;
}

namespace {
std::mutex g_dev_mu;
std::map<int, std::pair<int, int>> g_dev_props;               // device -> (SMs, opt-in smem)
std::map<std::pair<int, const void*>, size_t> g_smem_attr;    // (device, kernel) -> bytes set
int cur_device() {
    int d = 0;
    cudaGetDevice(&d);
    return d;
}
std::pair<int, int> dev_props() {
    const int d = cur_device();
    std::lock_guard<std::mutex> lk(g_dev_mu);
    auto it = g_dev_props.find(d);
    if (it != g_dev_props.end()) return it->second;
    int sms = 0, smem = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, d);
    cudaDeviceGetAttribute(&smem, cudaDevAttrMaxSharedMemoryPerBlockOptin, d);
    if (sms <= 0) sms = 148;
    if (smem <= 0) smem = 227 * 1024;
    g_dev_props[d] = {sms, smem};
    return {sms, smem};
}
}  // namespace

int dev_sms() { return dev_props().first; }
int dev_smem_optin() { return dev_props().second; }

cudaError_t ensure_smem_attr(const void* kernel, size_t bytes) {
    const int d = cur_device();
    std::lock_guard<std::mutex> lk(g_dev_mu);
    size_t& cur = g_smem_attr[{d, kernel}];
    if (bytes <= cur) return cudaSuccess;
    cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes);
    if (e == cudaSuccess) cur = bytes;
    return e;
}
}

// ====================================================================== C-ABI
extern "C" {

void rg_opts_default(rg_opts* o) {
    if (!o) return;
    o->panel = 0;
    o->precision = 0;
    o->nb = 32;
    o->scale = 1;
    o->reortho = -1;
    o->split = 0;
    o->sync = 1;
    o->solver = 0;
}

const char* rg_version(void) { return "rgsqr 0.1 sm_100a tcgen05/TMA"; }

const char* rg_status_string(int s) {
    if (s < 0) return "invalid argument";
    switch (s) {
        case RG_OK: return "ok";
        case RG_BREAKDOWN: return "breakdown: zero or non-finite column norm (rank deficient)";
        case RG_NOT_CONVERGED: return "not converged";
        case RG_NONFINITE: return "non-finite input";
        case RG_CUDA_ERROR: return "CUDA error";
        case RG_NCCL_ERROR: return "NCCL error";
        case RG_NO_DEVICE: return "no sm_100 CUDA device";
        case RG_ALLOC: return "allocation failed";
        default: return "unknown status";
    }
}

int rg_create(rg_handle* out, int device, void* stream) {
    if (!out) return -1;
    *out = nullptr;
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || device < 0 || device >= count) {
        cudaGetLastError();
        return RG_NO_DEVICE;
    }
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, device) != cudaSuccess || prop.major != 10) return RG_NO_DEVICE;
    if (cudaSetDevice(device) != cudaSuccess) return RG_NO_DEVICE;
    rg_handle h = new rg_handle_s();
    h->device = device;
    h->stream = reinterpret_cast<cudaStream_t>(stream);
    h->bind_bufs();
    if (cudaMallocHost(&h->status_host, 64) != cudaSuccess) {
        delete h;
        return RG_ALLOC;
    }
    if (cudaStreamCreateWithFlags(&h->capture_stream, cudaStreamNonBlocking) != cudaSuccess) {
        cudaFreeHost(h->status_host);
        delete h;
        return RG_CUDA_ERROR;
    }
    if (!ensure_encode()) {
        cudaFreeHost(h->status_host);
        delete h;
        return RG_CUDA_ERROR;
    }
    *out = h;
    return RG_OK;
}

int rg_set_stream(rg_handle h, void* stream) {
    if (!h) return -1;
    h->stream = reinterpret_cast<cudaStream_t>(stream);
    return RG_OK;
}

static void detach_comm(rg_handle h);

int rg_destroy(rg_handle h) {
    if (!h) return -1;
    cudaSetDevice(h->device);
    cudaStreamSynchronize(h->stream);
    for (auto& p : h->plans)
        if (p->exec) cudaGraphExecDestroy(p->exec);
    if (h->cgls_exec) cudaGraphExecDestroy(h->cgls_exec);
    for (DevBuf* b : h->bufs()) b->release();
    for (auto& e : h->ev_pool) {
        cudaEventDestroy(e.first);
        cudaEventDestroy(e.second);
    }
    detach_comm(h);
    if (h->status_host) cudaFreeHost(h->status_host);
    if (h->capture_stream) cudaStreamDestroy(h->capture_stream);
    if (h->cs_in) cudaStreamDestroy(h->cs_in);
    if (h->cs_out) cudaStreamDestroy(h->cs_out);
    for (auto e : h->pipe_ev) cudaEventDestroy(e);
    delete h;
    return RG_OK;
}

int64_t rg_last_info(rg_handle h) { return h ? h->last_info : -1; }

int64_t rg_last_launches(rg_handle h) { return h ? (int64_t)h->last_launches : -1; }

int rg_nccl_load(const char* path) {
    if (g_nccl.lib) return RG_OK;
    void* lib = dlopen(path ? path : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!lib) return RG_NCCL_ERROR;
    g_nccl.GetUniqueId = (decltype(g_nccl.GetUniqueId))dlsym(lib, "ncclGetUniqueId");
    g_nccl.CommInitRank = (decltype(g_nccl.CommInitRank))dlsym(lib, "ncclCommInitRank");
    g_nccl.CommDestroy = (decltype(g_nccl.CommDestroy))dlsym(lib, "ncclCommDestroy");
    g_nccl.AllReduce = (decltype(g_nccl.AllReduce))dlsym(lib, "ncclAllReduce");
    g_nccl.AllGather = (decltype(g_nccl.AllGather))dlsym(lib, "ncclAllGather");
    if (!g_nccl.GetUniqueId || !g_nccl.CommInitRank || !g_nccl.AllReduce || !g_nccl.AllGather) {
        dlclose(lib);
        return RG_NCCL_ERROR;
    }
    g_nccl.lib = lib;
    return RG_OK;
}

int rg_comm_unique_id(void* id128) {
    if (!id128) return -1;
    if (!g_nccl.lib && rg_nccl_load(nullptr) != RG_OK) return RG_NCCL_ERROR;
    ncclUniqueId id;
    if (g_nccl.GetUniqueId(&id) != ncclSuccess) return RG_NCCL_ERROR;
    memcpy(id128, &id, sizeof(id));
    return RG_OK;
}

// drop every cached plan / graph (their collectives and split decisions depend on the mode)
static void reset_plans(rg_handle h) {
    for (auto& p : h->plans)
        if (p->exec) cudaGraphExecDestroy(p->exec);
    h->plans.clear();
    if (h->cgls_exec) cudaGraphExecDestroy(h->cgls_exec);
    h->cgls_exec = nullptr;
    h->cgls_key[0] = nullptr;
}

static void detach_comm(rg_handle h) {
    if (h->comm && h->own_comm && g_nccl.CommDestroy) g_nccl.CommDestroy(h->comm);
    h->comm = nullptr;
    h->own_comm = false;
    if (h->vgroup) {
        std::lock_guard<std::mutex> lk(h->vgroup->mu);
        --h->vgroup->attached;
    }
    h->vgroup = nullptr;
    h->rank = 0;
    h->nranks = 1;
}

int rg_comm_init(rg_handle h, const void* id128, int rank, int nranks) {
    if (!h) return -1;
    if (!id128) return -2;
    if (nranks < 1 || nranks > RG_MAX_RANKS) return -4;
    if (rank < 0 || rank >= nranks) return -3;
    if (!g_nccl.lib && rg_nccl_load(nullptr) != RG_OK) return RG_NCCL_ERROR;
    ncclUniqueId id;
    memcpy(&id, id128, sizeof(id));
    cudaSetDevice(h->device);
    ncclComm_t c = nullptr;
    if (g_nccl.CommInitRank(&c, nranks, id, rank) != ncclSuccess) return RG_NCCL_ERROR;
    detach_comm(h);
    h->comm = c;
    h->own_comm = true;
    h->rank = rank;
    h->nranks = nranks;
    reset_plans(h);
    return RG_OK;
}

int rg_set_comm(rg_handle h, void* nccl_comm, int rank, int nranks) {
    if (!h) return -1;
    if (nccl_comm && (nranks < 1 || nranks > RG_MAX_RANKS)) return -4;
    if (nccl_comm && (rank < 0 || rank >= nranks)) return -3;
    if (nccl_comm && !g_nccl.lib && rg_nccl_load(nullptr) != RG_OK) return RG_NCCL_ERROR;
    detach_comm(h);
    if (nccl_comm) {
        h->comm = reinterpret_cast<ncclComm_t>(nccl_comm);
        h->own_comm = false;
        h->rank = rank;
        h->nranks = nranks;
    }
    reset_plans(h);
    return RG_OK;
}

int rg_vgroup_create(void** group, int nranks) {
    if (!group) return -1;
    *group = nullptr;
    if (nranks < 1 || nranks > RG_MAX_RANKS) return -2;
    VGroup* g = new VGroup();
    g->P = nranks;
    g->slots.resize(nranks);
    g->ready.resize(nranks, nullptr);
    for (int r = 0; r < nranks; ++r)
        if (cudaEventCreateWithFlags(&g->ready[r], cudaEventDisableTiming) != cudaSuccess) return RG_CUDA_ERROR;
    if (cudaEventCreateWithFlags(&g->done, cudaEventDisableTiming) != cudaSuccess) return RG_CUDA_ERROR;
    if (cudaMalloc(&g->dptrs, sizeof(void*) * RG_MAX_RANKS) != cudaSuccess) return RG_ALLOC;
    cudaGetDevice(&g->device);
    *group = g;
    return RG_OK;
}

int rg_vgroup_destroy(void* group) {
    VGroup* g = reinterpret_cast<VGroup*>(group);
    if (!g) return -1;
    {
        std::lock_guard<std::mutex> lk(g->mu);
        if (g->attached > 0) return -1;   // detach (rg_set_vcomm(h, NULL, 0) / rg_destroy) first
    }
    cudaDeviceSynchronize();
    for (auto e : g->ready) cudaEventDestroy(e);
    cudaEventDestroy(g->done);
    if (g->scratch) cudaFree(g->scratch);
    if (g->dptrs) cudaFree(g->dptrs);
    delete g;
    return RG_OK;
}

int rg_set_vcomm(rg_handle h, void* group, int rank) {
    if (!h) return -1;
    VGroup* g = reinterpret_cast<VGroup*>(group);
    if (g && (rank < 0 || rank >= g->P)) return -3;
    if (g && g->device != h->device) return -2;
    detach_comm(h);
    if (g) {
        std::lock_guard<std::mutex> lk(g->mu);
        ++g->attached;
        h->vgroup = g;
        h->rank = rank;
        h->nranks = g->P;
    }
    reset_plans(h);
    return RG_OK;
}

int rg_debug_gaussian(rg_handle h, int64_t n, uint64_t seed, double* out) {
    if (!h) return -1;
    if (n < 0) return -2;
    if (!out || ptr_side(out) != SIDE_DEVICE) return -4;
    cudaSetDevice(h->device);
    RG_CUDA(rg::launch_gaussian_philox(n, seed, out, nullptr, h->stream));
    RG_CUDA(cudaStreamSynchronize(h->stream));
    return RG_OK;
}

int rg_debug_philox(rg_handle h, int64_t ncalls, uint64_t seed, uint32_t* words) {
    if (!h) return -1;
    if (ncalls < 0) return -2;
    if (!words || ptr_side(words) != SIDE_DEVICE) return -4;
    cudaSetDevice(h->device);
    RG_CUDA(rg::launch_philox_words(ncalls, seed, words, h->stream));
    RG_CUDA(cudaStreamSynchronize(h->stream));
    return RG_OK;
}

int rg_profile_enable(rg_handle h, int enable) {
    if (!h) return -1;
    h->prof = enable != 0;
    return RG_OK;
}
int rg_profile_reset(rg_handle h) {
    if (!h) return -1;
    prof_collect(h);
    for (int i = 0; i < PC_N; ++i) {
        h->prof_ms[i] = 0;
        h->prof_launches[i] = 0;
        h->prof_flops[i] = 0;
        h->prof_bytes[i] = 0;
    }
    return RG_OK;
}
int rg_profile_get(rg_handle h, int cls, double* ms, int64_t* launches, double* flops, double* bytes) {
    if (!h) return -1;
    if (cls < 0 || cls >= PC_N) return -2;
    prof_collect(h);
    if (ms) *ms = h->prof_ms[cls];
    if (launches) *launches = h->prof_launches[cls];
    if (flops) *flops = h->prof_flops[cls];
    if (bytes) *bytes = h->prof_bytes[cls];
    return RG_OK;
}

// rgsqr_factor on pinned host buffers, one pass: column-chunked H2D of A on cs_in, the plan
// enqueued eagerly with a wait per chunk (HostPipe), Q columns D2H on cs_out as their panels
// finish (with the matching columns of R, unscaled piecewise); the user's stream joins cs_out
// before the status check.
int factor_host_pipelined(rg_handle h, int64_t m, int64_t n, const float* A, int64_t lda, float* Q, int64_t ldq,
                          float* R, int64_t ldr, const rg_opts& o) {
    if (!h->stageQ.ensure((size_t)m * n * 4) || !h->stageR.ensure((size_t)n * n * 4)) return RG_ALLOC;
    if (!h->cs_in) RG_CUDA(cudaStreamCreateWithFlags(&h->cs_in, cudaStreamNonBlocking));
    if (!h->cs_out) RG_CUDA(cudaStreamCreateWithFlags(&h->cs_out, cudaStreamNonBlocking));
    HostPipe pp;
    pp.chunk = 128;
    const int nchunks = (int)((n + pp.chunk - 1) / pp.chunk);
    while ((int)h->pipe_ev.size() < 3 + nchunks) {
        cudaEvent_t e;
        RG_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
        h->pipe_ev.push_back(e);
    }
    std::vector<cudaEvent_t> in_ev(h->pipe_ev.begin() + 3, h->pipe_ev.begin() + 3 + nchunks);
    float* dQ = h->stageQ.as<float>();
    float* dR = h->stageR.as<float>();
    cudaStream_t st = h->stream;
    // the staging buffer is free once everything before this call on the user's stream is done
    RG_CUDA(cudaEventRecord(h->pipe_ev[1], st));
    RG_CUDA(cudaStreamWaitEvent(h->cs_in, h->pipe_ev[1], 0));
    RG_CUDA(cudaStreamWaitEvent(h->cs_out, h->pipe_ev[1], 0));
    for (int k = 0; k < nchunks; ++k) {
        const int64_t c = (int64_t)k * pp.chunk, nc = std::min<int64_t>(pp.chunk, n - c);
        RG_CUDA(cudaMemcpy2DAsync(dQ + c * m, m * 4, A + c * lda, lda * 4, m * 4, nc, cudaMemcpyHostToDevice,
                                  h->cs_in));
        RG_CUDA(cudaEventRecord(in_ev[k], h->cs_in));
    }
    pp.hQ = Q;
    pp.hldq = ldq;
    pp.hR = R;
    pp.hldr = ldr;
    pp.in_ev = &in_ev;
    pp.cs_out = h->cs_out;
    pp.ev = h->pipe_ev[0];
    int rc = run_rgsqr(h, m, n, dQ, m, dQ, m, dR, n, o, o.split, false, &pp);
    // join both copy streams (also on error: nothing may still be in flight into the staging buffer)
    RG_CUDA(cudaEventRecord(h->pipe_ev[2], h->cs_out));
    RG_CUDA(cudaStreamWaitEvent(st, h->pipe_ev[2], 0));
    RG_CUDA(cudaEventRecord(h->pipe_ev[2], h->cs_in));
    RG_CUDA(cudaStreamWaitEvent(st, h->pipe_ev[2], 0));
    if (rc) {
        cudaStreamSynchronize(st);
        return rc;
    }
    return check_status(h);
}

int rgsqr_factor(rg_handle h, int64_t m_local, int64_t n, const float* A, int64_t lda, float* Q, int64_t ldq,
                 float* R, int64_t ldr, const rg_opts* opts) {
    if (!h) return -1;
    rg_opts o;
    if (opts) o = *opts; else rg_opts_default(&o);
    o.scale = o.scale ? 1 : 0;   // (-1 is the internal in-place reortho form)
    if (m_local < 1 || (h->nranks <= 1 && m_local < n)) return -2;
    if (n < 1 || n > 65535) return -3;
    if (!A) return -4;
    if (lda < m_local) return -5;
    if (!Q) return -6;
    if (ldq < m_local) return -7;
    if (!R) return -8;
    if (ldr < n) return -9;
    if (o.precision != 0 && o.precision != 1) return -10;
    cudaSetDevice(h->device);
    begin_call(h);
    const bool host = ptr_side(A) == SIDE_HOST;
    if (host && (ptr_side(Q) != SIDE_HOST || ptr_side(R) != SIDE_HOST)) return -6;
    const float* dA = A;
    float* dQ = Q;
    float* dR = R;
    int64_t dlda = lda, dldq = ldq, dldr = ldr;
    if (host && o.reortho <= 0 && h->nranks <= 1 && !h->prof && is_pinned(A) && is_pinned(Q) && is_pinned(R) &&
        getenv("RGSQR_NO_PIPE") == nullptr) {
        int rc = factor_host_pipelined(h, m_local, n, A, lda, Q, ldq, R, ldr, o);
        end_call(h);
        prof_collect(h);
        return rc;
    }
    if (host) {
        // stage: A -> device Q buffer (factor in place), results copied back
        if (!h->stageQ.ensure((size_t)m_local * n * 4) || !h->stageR.ensure((size_t)n * n * 4)) return RG_ALLOC;
        dQ = h->stageQ.as<float>();
        dR = h->stageR.as<float>();
        dldq = m_local;
        dldr = n;
        RG_CUDA(cudaMemcpy2DAsync(dQ, m_local * 4, A, lda * 4, m_local * 4, n, cudaMemcpyHostToDevice, h->stream));
        dA = dQ;
        dlda = m_local;
    }
    int rc = RG_OK;
    int passes = 1 + std::max(0, o.reortho);
    for (int p = 0; p < passes && rc == RG_OK; ++p) {
        if (p == 0) {
            rc = run_rgsqr(h, m_local, n, dA, dlda, dQ, dldq, dR, dldr, o, o.split);
        } else {
            // refinement pass: [Q2, R2] = RGSQR(Q) in split precision, R <- R2 R
            if (!h->aux.ensure((size_t)2 * n * n * 4)) return RG_ALLOC;
            float* R2 = h->aux.as<float>();
            float* Rt = R2 + n * n;
            if (rc == RG_OK && o.sync) rc = check_status(h);
            if (rc) break;
            rc = run_rgsqr(h, m_local, n, dQ, dldq, dQ, dldq, R2, n, o, 1);
            if (rc) break;
            RG_CUDA(rg::launch_trmm_upper(R2, n, dR, dldr, Rt, n, (int)n, h->stream));
            RG_CUDA(cudaMemcpy2DAsync(dR, dldr * 4, Rt, n * 4, n * 4, n, cudaMemcpyDeviceToDevice, h->stream));
        }
    }
    if (rc) return rc;
    if (host) {
        RG_CUDA(cudaMemcpy2DAsync(Q, ldq * 4, dQ, dldq * 4, m_local * 4, n, cudaMemcpyDeviceToHost, h->stream));
        RG_CUDA(cudaMemcpy2DAsync(R, ldr * 4, dR, dldr * 4, n * 4, n, cudaMemcpyDeviceToHost, h->stream));
    }
    if (o.sync || host) rc = check_status(h);
    if (getenv("RGSQR_LEAF_STATS") && h->cq_ws.p) {   // development: leaf-kernel counters so far
        unsigned long long c[3] = {0, 0, 0};
        cudaMemcpyAsync(c, h->cq_ws.as<double>() + rg::leaf_stats_offset(), sizeof(c), cudaMemcpyDeviceToHost,
                        h->stream);
        cudaStreamSynchronize(h->stream);
        fprintf(stderr, "[rgsqr leaf] launches %llu fast-Gram fallbacks %llu CholQR passes %llu\n", c[0], c[1], c[2]);
    }
    end_call(h);
    prof_collect(h);
    return rc;
}


int orthogonalize(rg_handle h, int64_t m_local, int64_t n, float* A, int64_t lda, float* R, int64_t ldr,
                  double orth_tol, int max_passes, int* passes_out, double* orth_est_out, const rg_opts* opts) {
    if (!h) return -1;
    rg_opts o;
    if (opts) o = *opts; else rg_opts_default(&o);
    o.scale = o.scale ? 1 : 0;   // (-1 is the internal in-place reortho form)
    if (m_local < 1 || (h->nranks <= 1 && m_local < n)) return -2;
    if (n < 1 || n > 65535) return -3;
    if (!A) return -4;
    if (lda < m_local) return -5;
    if (R && ldr < n) return -7;
    if (max_passes < 1) return -9;
    cudaSetDevice(h->device);
    begin_call(h);
    const bool host = ptr_side(A) == SIDE_HOST;
    float* dA = A;
    int64_t dlda = lda;
    if (host) {
        if (!h->stageQ.ensure((size_t)m_local * n * 4)) return RG_ALLOC;
        dA = h->stageQ.as<float>();
        dlda = m_local;
        RG_CUDA(cudaMemcpy2DAsync(dA, m_local * 4, A, lda * 4, m_local * 4, n, cudaMemcpyHostToDevice, h->stream));
    }
    if (!h->stageR.ensure((size_t)n * n * 4 + 256)) return RG_ALLOC;
    float* dR = h->stageR.as<float>();   // accumulated R (n x n, ld n)
    // tall blocks (n <= 256, too tall for the on-chip leaf): CholQR passes on the tensor cores
    // (reading #33), each falling back to the RGSQR pass when its kappa test fails
    bool tall = tall_wanted(h, m_local, n, dA, dlda);
    bool tall_ok = false;
    int rc = RG_OK;
    if (h->dist()) {   // the ranks' row counts differ: take the path only if every rank wants it
        if (!h->tallws.ensure(rg::tall_ws_bytes())) return RG_ALLOC;
        double* v = rg::tall_kout(h->tallws.p) + 3;
        const double mine = tall ? 1.0 : 0.0;
        RG_CUDA(cudaMemcpyAsync(v, &mine, sizeof(double), cudaMemcpyHostToDevice, h->stream));
        rc = nccl_allreduce(h, v, 1, ncclFloat64);
        if (rc) return rc;
        double all = 0;
        RG_CUDA(cudaMemcpyAsync(&all, v, sizeof(double), cudaMemcpyDeviceToHost, h->stream));
        RG_CUDA(cudaStreamSynchronize(h->stream));
        tall = all > h->nranks - 0.5;
    }
    if (tall) {
        if (!h->status.ensure(64)) return RG_ALLOC;
        rc = reset_status(h);
        if (rc == RG_OK) rc = tall_gram(h, m_local, (int)n, dA, dlda, true);
        if (rc == RG_OK) rc = tall_chol_apply(h, m_local, (int)n, dA, dlda, dR, n, true, &tall_ok);
    }
    if (rc == RG_OK && !tall_ok) rc = run_rgsqr(h, m_local, n, dA, dlda, dA, dlda, dR, n, o, o.split);
    int passes = 1;
    double est = -1.0;
    while (rc == RG_OK && passes < max_passes) {
        if (o.sync || orth_tol > 0) {
            rc = check_status(h);
            if (rc) break;
        }
        // A first pass with 16-bit GEMMs cannot be orthogonal below ~0.5 u16 n / sqrt(m) (reading
        // #9, SURVEY [EMU]): when a quarter of that floor is above the tolerance the probe after
        // pass 1 is skipped (the second pass runs anyway; only the estimate's cost is saved).
        const double u16 = o.precision ? 0x1p-8 : 0x1p-11;
        const double m_all = (double)m_local * std::max(1, h->nranks);
        const bool skip_probe = passes == 1 && !tall_ok && 0.25 * u16 * (double)n / std::sqrt(m_all) > orth_tol;
        // tall: the Gram of the current Q is the next pass's Gram and gives ||I - Q^T Q||_F exactly
        // (in its precision), so it replaces the Hutchinson probe
        if (tall) {
            rc = tall_gram(h, m_local, (int)n, dA, dlda, false);
            if (rc == RG_OK) rc = tall_orth(h, (int)n, &est);
            if (rc || (orth_tol > 0 && est <= orth_tol)) break;
        } else if (orth_tol > 0 && !skip_probe) {
            rc = orth_estimate(h, dA, dlda, m_local, (int)n, &est);
            if (rc || est <= orth_tol) break;
        }
        // [Q2, R2] = RGSQR(Q) with split-precision GEMMs (reading #9); R <- R2 R
        if (!h->lsR.ensure((size_t)n * n * 4 + 256)) return RG_ALLOC;
        float* R2 = h->lsR.as<float>();
        rg_opts o2 = o;
        o2.scale = -1;   // in place, unscaled (reading #32)
        bool ok2 = false;
        if (tall) rc = tall_chol_apply(h, m_local, (int)n, dA, dlda, R2, n, false, &ok2);
        if (rc == RG_OK && !ok2) rc = run_rgsqr(h, m_local, n, dA, dlda, dA, dlda, R2, n, o2, 1);
        if (rc) break;
        rc = trmm_into(h, R2, n, dR, n, (int)n);
        ++passes;
        est = -1.0;
    }
    if (rc) return rc;
    if (o.sync || host || orth_tol > 0 || orth_est_out) rc = check_status(h);
    if (rc) return rc;
    if ((orth_tol > 0 || orth_est_out) && est < 0) {
        rc = tall ? tall_gram(h, m_local, (int)n, dA, dlda, false) : orth_estimate(h, dA, dlda, m_local, (int)n, &est);
        if (rc == RG_OK && tall) rc = tall_orth(h, (int)n, &est);
        if (rc) return rc;
    }
    if (R) RG_CUDA(cudaMemcpy2DAsync(R, ldr * 4, dR, n * 4, n * 4, n,
                                     host ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice, h->stream));
    if (host)
        RG_CUDA(cudaMemcpy2DAsync(A, lda * 4, dA, dlda * 4, m_local * 4, n, cudaMemcpyDeviceToHost, h->stream));
    if (host || o.sync) RG_CUDA(cudaStreamSynchronize(h->stream));
    if (passes_out) *passes_out = passes;
    if (orth_est_out) *orth_est_out = est;
    end_call(h);
    prof_collect(h);
    if (orth_tol > 0 && est > orth_tol) return RG_NOT_CONVERGED;
    return RG_OK;
}

int ls_solve_refined(rg_handle h, int64_t m_local, int64_t n, const float* A, int64_t lda, const float* b, double* x,
                     double tol, int maxit, int* iters_out, double* relres_out, const rg_opts* opts) {
    if (!h) return -1;
    rg_opts o;
    if (opts) o = *opts; else rg_opts_default(&o);
    o.scale = o.scale ? 1 : 0;   // (-1 is the internal in-place reortho form)
    if (m_local < 1 || (h->nranks <= 1 && m_local < n)) return -2;
    if (n < 1 || n > 16384) return -3;
    if (!A) return -4;
    if (lda < m_local) return -5;
    if (!b) return -6;
    if (!x) return -7;
    if (!(tol >= 0)) return -8;
    if (maxit < 0) return -9;
    cudaSetDevice(h->device);
    begin_call(h);
    const bool host = ptr_side(A) == SIDE_HOST;
    const float* dA = A;
    const float* db = b;
    int64_t dlda = lda;
    if (host) {
        if (!h->stageA.ensure((size_t)m_local * n * 4) || !h->stageB.ensure((size_t)m_local * 4 + 64)) return RG_ALLOC;
        RG_CUDA(cudaMemcpy2DAsync(h->stageA.p, m_local * 4, A, lda * 4, m_local * 4, n, cudaMemcpyHostToDevice,
                                  h->stream));
        RG_CUDA(cudaMemcpyAsync(h->stageB.p, b, m_local * 4, cudaMemcpyHostToDevice, h->stream));
        dA = h->stageA.as<float>();
        db = h->stageB.as<float>();
        dlda = m_local;
    }
    // ---- QR preconditioner (reading #8): by default ONE RGSQR pass with split-precision (3 x 16-bit)
    // K1 / K2 -- its R makes kappa(A R^-1) ~ 1 + O(u32 kappa(A)), so CGLS converges in a few
    // iterations (config 3: 8, one QR pass, 6.5 ms) where the 16-bit pass + a reortho pass leaves
    // kappa(A R^-1) ~ 1.8 (19 iterations, two QR passes, 11.4 ms); opts->reortho >= 0 selects
    // RGSQR (+ that many reortho passes) in opts->split precision
    if (!h->lsQ.ensure((size_t)m_local * n * 4) || !h->stageR.ensure((size_t)n * n * 4 + 256)) return RG_ALLOC;
    float* Qw = h->lsQ.as<float>();
    float* Rw = h->stageR.as<float>();
    const int extra = o.reortho < 0 ? 0 : o.reortho;
    if (o.reortho < 0) o.split = 1;
    int rc = factor_with_reortho(h, m_local, n, dA, dlda, Qw, m_local, Rw, n, o, extra);
    if (rc) return rc;
    rc = check_status(h);
    if (rc) return rc;
    // ---- explicit R^{-1} (fp64)
    if (!h->rinv.ensure((size_t)2 * n * n * 8 + 64)) return RG_ALLOC;   // Rinv + its row-major copy
    RG_CUDA(rg::launch_trinv_upper(Rw, n, (int)n, h->rinv.as<double>(), h->stream));
    // ---- CGLS state: sc[16] | x p s t sv (n each) | r q (m each) | gemv work
    const size_t work = std::max({rg::gemv_n_work_doubles(m_local, (int)n), rg::gemv_t_work_doubles(m_local, (int)n),
                                  rg::gemv_nt_work_doubles((int)n) + (size_t)n});
    if (!h->cg.ensure((16 + 6 * (size_t)n + 2 * (size_t)m_local + work + 2048) * 8 + 256)) return RG_ALLOC;   // (LSQR: 6 n-vectors)
    double* base = h->cg.as<double>();
    double* sc = base;
    double* xd = sc + 16;
    double* p = xd + n;
    double* s = p + n;
    double* sv = s + 2 * n;
    double* r = sv + n;
    double* wk = r + 2 * m_local;
    const bool lsqr = o.solver == 1;
    // the one-pass product (CGLS and LSQR) needs 16 B aligned columns; the ranks' shards may differ, so under
    // dist every rank takes it only if all can (the two forms issue different allreduces)
    h->cgls_one_pass = rg::gemv_nt_ok(dA, dlda, (int)n);
    if (h->dist()) {
        const double mine = h->cgls_one_pass ? 1.0 : 0.0;
        RG_CUDA(cudaMemcpyAsync(sc + 10, &mine, sizeof(double), cudaMemcpyHostToDevice, h->stream));
        rc = nccl_allreduce(h, sc + 10, 1, ncclFloat64);
        if (rc) return rc;
        double all = 0;
        RG_CUDA(cudaMemcpyAsync(&all, sc + 10, sizeof(double), cudaMemcpyDeviceToHost, h->stream));
        RG_CUDA(cudaStreamSynchronize(h->stream));
        h->cgls_one_pass = all > h->nranks - 0.5;
    }
    {
        double init[16] = {0};
        init[8] = tol;
        RG_CUDA(cudaMemcpyAsync(sc, init, sizeof(init), cudaMemcpyHostToDevice, h->stream));
    }
    if (lsqr) {
        // LSQR start: u = b, beta_1 = |b|, p = R^-T A^T u, alpha_1 v_1 = p / beta_1, w = v, y = 0
        double* y = sc + 16;
        double* v = y + n;
        double* w = v + n;
        double* t = w + n;
        double* svl = t + n;
        double* pl = svl + n;
        double* u = pl + n;
        double* wkl = u + 2 * m_local;
        RG_CUDA(rg::launch_cgls_init(db, m_local, (int)n, u, y, h->stream));
        RG_CUDA(rg::launch_sqnorm(u, m_local, sc, 1, h->stream));
        rc = nccl_allreduce(h, sc + 1, 1, ncclFloat64);
        if (rc) return rc;
        RG_CUDA(rg::launch_gemv_t(dA, dlda, m_local, (int)n, u, svl, wkl, nullptr, h->stream));
        rc = nccl_allreduce(h, svl, n, ncclFloat64);
        if (rc) return rc;
        RG_CUDA(rg::launch_trmv(h->rinv.as<double>(), (int)n, svl, pl, 1, nullptr, h->stream));
        RG_CUDA(rg::launch_lsqr_step(pl, v, w, y, (int)n, sc, 1, h->stream));
    } else {
    RG_CUDA(rg::launch_cgls_init(db, m_local, (int)n, r, xd, h->stream));          // lines 4-5
    RG_CUDA(rg::launch_gemv_t(dA, dlda, m_local, (int)n, r, sv, wk, nullptr, h->stream));
    rc = nccl_allreduce(h, sv, n, ncclFloat64);
    if (rc) return rc;
    RG_CUDA(rg::launch_trmv(h->rinv.as<double>(), (int)n, sv, s, 1, nullptr, h->stream));  // line 6 (corrected)
    RG_CUDA(rg::launch_cgls_p(s, p, (int)n, sc, 1, h->stream));                    // lines 7-9
    }
    // ---- iterations in captured blocks of `blk`, convergence flag read between blocks
    const int blk = 8;
    int done_iters = 0;
    double hsc[16];
    const bool use_graph = !h->prof && !h->vgroup && getenv("RGSQR_NO_GRAPH") == nullptr;
    while (done_iters < maxit) {
        const int cnt = std::min(blk, maxit - done_iters);
        if (use_graph && cnt == blk) {
            const bool same = h->cgls_exec && h->cgls_key[0] == dA && h->cgls_key[1] == base &&
                              h->cgls_key[2] == h->rinv.p && h->cgls_key_mn[0] == m_local && h->cgls_key_mn[1] == n &&
                              h->cgls_key_mn[2] == dlda && h->cgls_solver == o.solver &&
                              h->cgls_graph_one_pass == h->cgls_one_pass;
            if (!same) {
                if (h->cgls_exec) cudaGraphExecDestroy(h->cgls_exec);
                h->cgls_exec = nullptr;
                cudaGraph_t g;
                cudaStream_t user = h->stream;
                h->stream = h->capture_stream;
                RG_CUDA(cudaStreamBeginCapture(h->stream, cudaStreamCaptureModeThreadLocal));
                const long long before = rg::g_launches;
                rc = lsqr ? enqueue_lsqr_iters(h, dA, dlda, m_local, (int)n, blk, base)
                          : enqueue_cgls_iters(h, dA, dlda, m_local, (int)n, blk, base);
                h->cgls_solver = o.solver;
                h->cgls_graph_one_pass = h->cgls_one_pass;
                const long long captured = rg::g_launches - before;
                rg::g_launches = before;
                h->cgls_key_mn[2] = dlda;
                cudaError_t ce = cudaStreamEndCapture(h->stream, &g);
                h->stream = user;
                if (rc) return rc;
                RG_CUDA(ce);
                cudaError_t ie = cudaGraphInstantiate(&h->cgls_exec, g, 0);
                cudaGraphDestroy(g);
                RG_CUDA(ie);
                h->cgls_key[0] = dA;
                h->cgls_key[1] = base;
                h->cgls_key[2] = h->rinv.p;
                h->cgls_key_mn[0] = m_local;
                h->cgls_key_mn[1] = n;
                h->cgls_key[3] = (const void*)(intptr_t)captured;
            }
            RG_CUDA(cudaGraphLaunch(h->cgls_exec, h->stream));
            h->replayed += (long long)(intptr_t)h->cgls_key[3];
        } else {
            const long long before = rg::g_launches;
            rc = lsqr ? enqueue_lsqr_iters(h, dA, dlda, m_local, (int)n, cnt, base)
                      : enqueue_cgls_iters(h, dA, dlda, m_local, (int)n, cnt, base);
            if (rc) return rc;
        }
        done_iters += cnt;
        RG_CUDA(cudaMemcpyAsync(hsc, sc, sizeof(hsc), cudaMemcpyDeviceToHost, h->stream));
        RG_CUDA(cudaStreamSynchronize(h->stream));
        if (hsc[6] != 0.0) break;
    }
    if (done_iters == 0) {
        RG_CUDA(cudaMemcpyAsync(hsc, sc, sizeof(hsc), cudaMemcpyDeviceToHost, h->stream));
        RG_CUDA(cudaStreamSynchronize(h->stream));
    }
    if (lsqr) {   // x = R^-1 y (y lives where CGLS keeps x)
        double* y = sc + 16;
        double* tt = y + 3 * n;
        RG_CUDA(rg::launch_trmv(h->rinv.as<double>(), (int)n, y, tt, 0, nullptr, h->stream));
        RG_CUDA(cudaMemcpyAsync(y, tt, n * 8, cudaMemcpyDeviceToDevice, h->stream));
    }
    RG_CUDA(cudaMemcpyAsync(x, xd, n * 8, host ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice, h->stream));
    RG_CUDA(cudaStreamSynchronize(h->stream));
    if (iters_out) *iters_out = (int)hsc[7];
    if (relres_out) *relres_out = hsc[4] > 0 ? hsc[5] / hsc[4] : 0.0;
    end_call(h);
    prof_collect(h);
    if (!(hsc[6] != 0.0) && maxit > 0 && !(hsc[5] <= tol * hsc[4])) return RG_NOT_CONVERGED;
    return RG_OK;
}


int lowrank_approx(rg_handle h, int64_t m_local, int64_t n, const float* A, int64_t lda, int rank, int oversample,
                   int power_iters, uint64_t seed, float* U, int64_t ldu, float* S, float* V, int64_t ldv,
                   const rg_opts* opts) {
    if (!h) return -1;
    rg_opts o;
    if (opts) o = *opts; else rg_opts_default(&o);
    o.scale = o.scale ? 1 : 0;   // (-1 is the internal in-place reortho form)
    if (m_local < 1) return -2;
    if (n < 1 || n > 65535) return -3;
    if (!A) return -4;
    if (lda < m_local) return -5;
    const int l = rank + oversample;
    if (rank < 1 || oversample < 0 || l > n || (h->nranks <= 1 && l > m_local)) return rank < 1 ? -6 : -7;
    if (power_iters < 0) return -8;
    if (!U) return -10;
    if (ldu < m_local) return -11;
    if (!S) return -12;
    if (!V) return -13;
    if (ldv < n) return -14;
    cudaSetDevice(h->device);
    begin_call(h);
    cudaStream_t st = h->stream;
    const bool host = ptr_side(A) == SIDE_HOST;
    const float* dA = A;
    int64_t dlda = lda;
    float *dU = U, *dS = S, *dV = V;
    int64_t dldu = ldu, dldv = ldv;
    if (host) {
        if (!h->stageA.ensure((size_t)m_local * n * 4) || !h->stageQ.ensure((size_t)m_local * rank * 4) ||
            !h->stageR.ensure(((size_t)n * rank + rank) * 4 + 256))
            return RG_ALLOC;
        RG_CUDA(cudaMemcpy2DAsync(h->stageA.p, m_local * 4, A, lda * 4, m_local * 4, n, cudaMemcpyHostToDevice, st));
        dA = h->stageA.as<float>();
        dlda = m_local;
        dU = h->stageQ.as<float>();
        dldu = m_local;
        dV = h->stageR.as<float>();
        dldv = n;
        dS = dV + (size_t)n * rank;
    }
    const int bf = o.precision;
    const int64_t ldm16 = round_up(std::max<int64_t>(m_local, 8), 8);
    const int64_t ldn16 = round_up(std::max<int64_t>(n, 8), 8);
    const int64_t ldl16 = round_up(std::max(l, 8), 8);
    bool ok = h->lrA16.ensure((size_t)ldm16 * n * 2) && h->lrB16.ensure((size_t)ldn16 * l * 2) &&
              h->lrB16l.ensure((size_t)ldl16 * rank * 2 + 64) && h->lrY.ensure((size_t)m_local * l * 4) &&
              h->lrZ.ensure((size_t)n * l * 4) && h->lrQ16.ensure((size_t)std::max(ldm16, ldn16) * l * 2) &&
              h->lrQ16l.ensure((size_t)std::max(ldm16, ldn16) * l * 2) && h->lrR.ensure((size_t)l * l * 4) &&
              h->lrW.ensure(rg::jacobi_w_doubles(l) * 8) && h->lrV.ensure((size_t)l * l * 8) &&
              h->lrUb.ensure((size_t)l * l * 4) && h->lrVb.ensure((size_t)l * l * 4) && h->lrSig.ensure(l * 8 + 64) &&
              h->lrOm.ensure((size_t)n * l * 8) && h->lrScale.ensure(n * 4 + 64) && h->lrFlags.ensure(512) &&
              h->partial.ensure(rg::colnorm_partial_doubles(m_local, (int)n) * 8 + 64) && h->norm2.ensure(n * 8 + 64) &&
              h->status.ensure(64);
    if (!ok) return RG_ALLOC;
    uint16_t* A16 = h->lrA16.as<uint16_t>();
    float* sc = h->lrScale.as<float>();
    float* Y = h->lrY.as<float>();
    float* Z = h->lrZ.as<float>();
    float* Rl = h->lrR.as<float>();
    int rc = reset_status(h);
    if (rc) return rc;
    // ---- power-of-two column scaling of A into fp16 range (section 3.5): A16 = fp16(A P)
    RG_CUDA(rg::launch_colnorm(dA, dlda, m_local, (int)n, h->partial.as<double>(), h->norm2.as<double>(), st));
    if (h->dist()) {
        rc = nccl_allreduce(h, h->norm2.p, n, ncclFloat64);
        if (rc) return rc;
    }
    RG_CUDA(rg::launch_colscale(h->norm2.as<double>(), (int)n, 1, sc, h->status.as<int>(), 0, st));
    RG_CUDA(rg::launch_scale_cast(dA, dlda, nullptr, 0, A16, nullptr, ldm16, m_local, (int)n, sc, bf, st));
    // ---- sketch: Omega (n x l) ~ N(0,1) (Philox); B16 = fp16(P^{-1} Omega)
    RG_CUDA(rg::launch_gaussian_philox((int64_t)n * l, seed, h->lrOm.as<double>(), nullptr, st));
    RG_CUDA(rg::launch_cast_rows64(h->lrOm.as<double>(), n, n, l, sc, h->lrB16.as<uint16_t>(), nullptr, ldn16, bf, st));
    // Y = A Omega = (A P)(P^{-1} Omega)
    rc = gemm_nn(h, m_local, l, (int)n, A16, nullptr, ldm16, h->lrB16.as<uint16_t>(), nullptr, ldn16, Y, m_local, bf);
    if (rc) return rc;
    rg_opts qo = o;
    qo.sync = 0;
    auto project = [&](float* out) -> int {
        // out (n x l) = A^T Q with Q's fp16 image in the RGSQR workspace (ldh): (A P)^T Q / P
        int r2 = gemm_tn(h, m_local, (int)n, l, A16, ldm16, h->qh.as<uint16_t>(), round_up(std::max<int64_t>(m_local, 8), 8),
                         out, n, bf);
        if (r2) return r2;
        if (h->dist()) {
            r2 = nccl_allreduce(h, out, (size_t)n * l, ncclFloat32);
            if (r2) return r2;
        }
        RG_CUDA(rg::launch_unscale_rows(out, n, n, l, sc, st));
        return RG_OK;
    };
    for (int it = 0; it < power_iters; ++it) {
        rc = run_rgsqr(h, m_local, l, Y, m_local, Y, m_local, Rl, l, qo, 0);          // Q = qr(Y)
        if (rc) return rc;
        rc = project(Z);                                                            // Z = A^T Q
        if (rc) return rc;
        rc = run_rgsqr(h, n, l, Z, n, Z, n, Rl, l, qo, 0, true);                     // Q_z = qr(Z)
        if (rc) return rc;
        RG_CUDA(rg::launch_cast_rows(Z, n, n, l, sc, h->lrB16.as<uint16_t>(), nullptr, ldn16, bf, st));
        rc = gemm_nn(h, m_local, l, (int)n, A16, nullptr, ldm16, h->lrB16.as<uint16_t>(), nullptr, ldn16, Y, m_local,
                     bf);                                                           // Y = A Q_z
        if (rc) return rc;
    }
    rc = run_rgsqr(h, m_local, l, Y, m_local, Y, m_local, Rl, l, qo, 0);              // Q = qr(Y)
    if (rc) return rc;
    rc = project(Z);                                                                // B^T = A^T Q
    if (rc) return rc;
    rc = run_rgsqr(h, n, l, Z, n, Z, n, Rl, l, qo, 0, true);                         // B^T = Q_b R_b
    if (rc) return rc;
    // ---- R_b = U_b S V_b^T (one-sided Jacobi, fp64)
    RG_CUDA(rg::launch_jacobi_svd(Rl, l, l, rank, h->lrW.as<double>(), h->lrV.as<double>(), h->lrSig.as<double>(),
                                  h->lrFlags.as<int>(), dS, h->lrUb.as<float>(), h->lrVb.as<float>(), st));
    // ---- U = Q V_b(:, 1:r), V = Q_b U_b(:, 1:r)  (split-precision tensor-core products)
    uint16_t* q16 = h->lrQ16.as<uint16_t>();
    uint16_t* q16l = h->lrQ16l.as<uint16_t>();
    uint16_t* b16 = h->lrB16.as<uint16_t>();
    uint16_t* b16l = h->lrB16l.as<uint16_t>();
    RG_CUDA(rg::launch_cast_rows(Y, m_local, m_local, l, nullptr, q16, q16l, ldm16, bf, st));
    RG_CUDA(rg::launch_cast_rows(h->lrVb.as<float>(), l, l, rank, nullptr, b16, b16l, ldl16, bf, st));
    rc = gemm_nn(h, m_local, rank, l, q16, q16l, ldm16, b16, b16l, ldl16, dU, dldu, bf);
    if (rc) return rc;
    RG_CUDA(rg::launch_cast_rows(Z, n, n, l, nullptr, q16, q16l, ldn16, bf, st));
    RG_CUDA(rg::launch_cast_rows(h->lrUb.as<float>(), l, l, rank, nullptr, b16, b16l, ldl16, bf, st));
    rc = gemm_nn(h, n, rank, l, q16, q16l, ldn16, b16, b16l, ldl16, dV, dldv, bf);
    if (rc) return rc;
    if (host) {
        RG_CUDA(cudaMemcpy2DAsync(U, ldu * 4, dU, dldu * 4, m_local * 4, rank, cudaMemcpyDeviceToHost, st));
        RG_CUDA(cudaMemcpy2DAsync(V, ldv * 4, dV, dldv * 4, n * 4, rank, cudaMemcpyDeviceToHost, st));
        RG_CUDA(cudaMemcpyAsync(S, dS, rank * 4, cudaMemcpyDeviceToHost, st));
    }
    if (o.sync || host) rc = check_status(h);
    end_call(h);
    prof_collect(h);
    return rc;
}


// Deterministic QR-SVD low-rank approximation of a tall-skinny A (section 3.4, Table 4):
// A = Q R (one RGSQR pass: "the roundoff errors in RGSQRF is insignificant, thus no refinement or
// re-orthogonalization is needed"), R = U_R S V_R^T (one-sided Jacobi, fp64), and
// A_r = (Q U_R(:, 1:r)) S_r V_R(:, 1:r)^T.  U = Q U_R(:, 1:r) with the split-precision tensor-core
// product (reading #9); V = V_R(:, 1:r).
int lowrank_qrsvd(rg_handle h, int64_t m_local, int64_t n, const float* A, int64_t lda, int rank, float* U,
                  int64_t ldu, float* S, float* V, int64_t ldv, const rg_opts* opts) {
    if (!h) return -1;
    rg_opts o;
    if (opts) o = *opts; else rg_opts_default(&o);
    o.scale = o.scale ? 1 : 0;   // (-1 is the internal in-place reortho form)
    if (m_local < 1 || (h->nranks <= 1 && m_local < n)) return -2;
    if (n < 1 || n > 4096) return -3;
    if (!A) return -4;
    if (lda < m_local) return -5;
    if (rank < 1 || rank > n) return -6;
    if (!U) return -7;
    if (ldu < m_local) return -8;
    if (!S) return -9;
    if (!V) return -10;
    if (ldv < n) return -11;
    cudaSetDevice(h->device);
    begin_call(h);
    cudaStream_t st = h->stream;
    const bool host = ptr_side(A) == SIDE_HOST;
    const float* dA = A;
    int64_t dlda = lda;
    float *dU = U, *dS = S, *dV = V;
    int64_t dldu = ldu, dldv = ldv;
    if (host) {
        if (!h->stageA.ensure((size_t)m_local * n * 4) || !h->stageQ.ensure((size_t)m_local * rank * 4) ||
            !h->stageR.ensure(((size_t)n * rank + rank) * 4 + 256))
            return RG_ALLOC;
        RG_CUDA(cudaMemcpy2DAsync(h->stageA.p, m_local * 4, A, lda * 4, m_local * 4, n, cudaMemcpyHostToDevice, st));
        dA = h->stageA.as<float>();
        dlda = m_local;
        dU = h->stageQ.as<float>();
        dldu = m_local;
        dV = h->stageR.as<float>();
        dldv = n;
        dS = dV + (size_t)n * rank;
    }
    const int l = (int)n;
    const int64_t ldm16 = round_up(std::max<int64_t>(m_local, 8), 8);
    const int64_t ldl16 = round_up(std::max(l, 8), 8);
    bool ok = h->lsQ.ensure((size_t)m_local * n * 4) && h->lrR.ensure((size_t)l * l * 4) &&
              h->lrW.ensure(rg::jacobi_w_doubles(l) * 8) && h->lrV.ensure((size_t)l * l * 8) &&
              h->lrUb.ensure((size_t)l * l * 4) && h->lrVb.ensure((size_t)l * l * 4) && h->lrSig.ensure(l * 8 + 64) &&
              h->lrFlags.ensure(512) && h->lrQ16.ensure((size_t)ldm16 * l * 2) && h->lrQ16l.ensure((size_t)ldm16 * l * 2) &&
              h->lrB16.ensure((size_t)ldl16 * rank * 2 + 64) && h->lrB16l.ensure((size_t)ldl16 * rank * 2 + 64);
    if (!ok) return RG_ALLOC;
    float* Qw = h->lsQ.as<float>();
    float* Rl = h->lrR.as<float>();
    rg_opts qo = o;
    qo.sync = 0;
    int rc = run_rgsqr(h, m_local, n, dA, dlda, Qw, m_local, Rl, l, qo, 0);   // A = Q R
    if (rc) return rc;
    rc = check_status(h);
    if (rc) return rc;
    // R = U_R S V_R^T: Jacobi on R (trans = 0 in the grid form gives U_R = W S^-1, V_R = J)
    RG_CUDA(rg::launch_jacobi_svd(Rl, l, l, rank, h->lrW.as<double>(), h->lrV.as<double>(), h->lrSig.as<double>(),
                                  h->lrFlags.as<int>(), dS, h->lrUb.as<float>(), h->lrVb.as<float>(), st));
    // U = Q U_R(:, 1:r)  (split-precision tensor-core product, ~fp32 accurate)
    uint16_t* q16 = h->lrQ16.as<uint16_t>();
    uint16_t* q16l = h->lrQ16l.as<uint16_t>();
    uint16_t* b16 = h->lrB16.as<uint16_t>();
    uint16_t* b16l = h->lrB16l.as<uint16_t>();
    RG_CUDA(rg::launch_cast_rows(Qw, m_local, m_local, l, nullptr, q16, q16l, ldm16, o.precision, st));
    RG_CUDA(rg::launch_cast_rows(h->lrUb.as<float>(), l, l, rank, nullptr, b16, b16l, ldl16, o.precision, st));
    rc = gemm_nn(h, m_local, rank, l, q16, q16l, ldm16, b16, b16l, ldl16, dU, dldu, o.precision);
    if (rc) return rc;
    RG_CUDA(cudaMemcpy2DAsync(dV, dldv * 4, h->lrVb.as<float>(), (size_t)l * 4, (size_t)n * 4, rank,
                              cudaMemcpyDeviceToDevice, st));
    if (host) {
        RG_CUDA(cudaMemcpy2DAsync(U, ldu * 4, dU, dldu * 4, m_local * 4, rank, cudaMemcpyDeviceToHost, st));
        RG_CUDA(cudaMemcpy2DAsync(V, ldv * 4, dV, dldv * 4, n * 4, rank, cudaMemcpyDeviceToHost, st));
        RG_CUDA(cudaMemcpyAsync(S, dS, rank * 4, cudaMemcpyDeviceToHost, st));
    }
    if (o.sync || host) rc = check_status(h);
    end_call(h);
    prof_collect(h);
    return rc;
}

}  // extern "C"
