// mgpu.cu — the cross-GPU exchange and the multi-GPU / pipelined executor.
//
// No GPU in the paper (one C2070); BASELINE.json north_star part (4): "sharding of
// the cube along its outermost dimension across the 8 GPUs of one box, with each GPU reducing its
// slab and a single small NCCL allreduce/reduce of per-query partials over NVLink".  The partial
// format is olap.h's: sum (int64 wraparound / fp64 bits, combine +), MAX code and ~MIN code
// (int32, combine max).  One ncclGroup per batch carries both reductions for every device.
//
// NCCL is loaded at run time (dlopen of libnccl.so.2, or $OLAP_NCCL_LIB): a process that never
// shards a cube does not need it, and a process that already loaded torch's NCCL shares that copy.
// Every NCCL failure maps to OLAP_E_NCCL with NCCL's message; after each exchange the
// communicators' asynchronous error state is polled (ncclCommGetAsyncError) and a failed
// communicator is aborted and refuses further batches.
#include <dlfcn.h>
#include <nccl.h>

#include <cstring>
#include <mutex>
#include <vector>

#include "common.cuh"
#include "mgpu.h"

namespace olap {

// ------------------------------------------------------------------ NCCL, loaded at run time
namespace {

struct NcclApi {
    bool ok = false;
    std::string why;
    int version = 0;
    ncclResult_t (*GetVersion)(int*) = nullptr;
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommInitAll)(ncclComm_t*, int, const int*) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*CommAbort)(ncclComm_t) = nullptr;
    ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t*) = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    ncclResult_t (*Reduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, int, ncclComm_t,
                           cudaStream_t) = nullptr;
    ncclResult_t (*AllReduce)(const void*, void*, size_t, ncclDataType_t, ncclRedOp_t, ncclComm_t,
                              cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
};

NcclApi g_nccl;
std::once_flag g_nccl_once;

template <class F>
bool load_sym(void* h, const char* name, F& f) {
    f = reinterpret_cast<F>(dlsym(h, name));
    return f != nullptr;
}

void load_nccl() {
    const char* env = getenv("OLAP_NCCL_LIB");
    const char* names[] = {env, "libnccl.so.2", "libnccl.so"};
    void* h = nullptr;
    for (const char* n : names)
        if (n && (h = dlopen(n, RTLD_NOW | RTLD_GLOBAL))) break;
    if (!h) {
        const char* e = dlerror();
        g_nccl.why = std::string("cannot load NCCL (libnccl.so.2): ") + (e ? e : "?");
        return;
    }
    NcclApi& a = g_nccl;
    const bool ok = load_sym(h, "ncclGetVersion", a.GetVersion) && load_sym(h, "ncclGetUniqueId", a.GetUniqueId) &&
                    load_sym(h, "ncclCommInitRank", a.CommInitRank) && load_sym(h, "ncclCommInitAll", a.CommInitAll) &&
                    load_sym(h, "ncclCommDestroy", a.CommDestroy) && load_sym(h, "ncclCommAbort", a.CommAbort) &&
                    load_sym(h, "ncclCommGetAsyncError", a.CommGetAsyncError) &&
                    load_sym(h, "ncclGetErrorString", a.GetErrorString) && load_sym(h, "ncclReduce", a.Reduce) &&
                    load_sym(h, "ncclAllReduce", a.AllReduce) && load_sym(h, "ncclGroupStart", a.GroupStart) &&
                    load_sym(h, "ncclGroupEnd", a.GroupEnd);
    if (!ok) {
        a.why = "libnccl.so.2 lacks a required symbol";
        return;
    }
    a.GetVersion(&a.version);
    a.ok = true;
}

int nccl_api(const NcclApi** out) {
    std::call_once(g_nccl_once, load_nccl);
    if (!g_nccl.ok) return set_error(OLAP_E_NCCL, "%s", g_nccl.why.c_str());
    *out = &g_nccl;
    return OLAP_OK;
}

#define OLAP_NCCL_TRY(api, expr)                                                                            \
    do {                                                                                                    \
        ncclResult_t r_ = (expr);                                                                           \
        if (r_ != ncclSuccess)                                                                              \
            return ::olap::set_error(OLAP_E_NCCL, "%s failed: %s (%s:%d)", #expr, (api)->GetErrorString(r_), \
                                     __FILE__, __LINE__);                                                   \
    } while (0)

struct DevGuard {
    int prev = -1;
    bool ok = false;
    explicit DevGuard(int dev) {
        if (cudaGetDevice(&prev) == cudaSuccess && cudaSetDevice(dev) == cudaSuccess) ok = true;
    }
    ~DevGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};

}  // namespace
}  // namespace olap

// a communicator over the ranks that hold the shards of one cube (one process per GPU)
struct olap_comm {
    ncclComm_t comm = nullptr;
    int nranks = 0, rank = 0, device = 0;
    bool failed = false;
};

namespace olap {

namespace {

// poll a communicator after an exchange; abort it on an asynchronous error
int check_comm(const NcclApi* api, ncclComm_t comm, bool* failed) {
    ncclResult_t st = ncclSuccess;
    OLAP_NCCL_TRY(api, api->CommGetAsyncError(comm, &st));
    if (st != ncclSuccess && st != ncclInProgress) {
        *failed = true;
        api->CommAbort(comm);
        return set_error(OLAP_E_NCCL, "NCCL communicator failed asynchronously: %s (aborted)",
                         api->GetErrorString(st));
    }
    return OLAP_OK;
}

}  // namespace

// ------------------------------------------------------------------ executor

struct DevCtx {
    int device = 0;
    std::vector<olap_cube*> shards;
    ncclComm_t comm = nullptr;  // owned (group) or borrowed (olap_comm)
    cudaStream_t cs = nullptr;  // compute: inputs, partials, local combine
    cudaStream_t ms = nullptr;  // exchange: NCCL, finalize, results
    cudaEvent_t ev_in = nullptr, ev_part[2] = {}, ev_free[2] = {};
    olap_range* d_ranges[2] = {};
    int32_t* d_ops[2] = {};
    int64_t* acc_sum[2] = {};
    int32_t* acc_ext[2] = {};
    int64_t* tmp_sum = nullptr;
    int32_t* tmp_ext = nullptr;
    olap_result* d_res[2] = {};
};

struct Exec {
    int nd = 0, dtype = 0;
    int64_t n[8] = {};
    std::vector<DevCtx> dev;
    olap_comm* comm = nullptr;  // multi-process mode
    bool own_comms = false;     // group mode (reduce to devices[0])
    bool failed = false;
    const NcclApi* api = nullptr;
    int64_t cap = 0;
    char* h_pin = nullptr;  // [2] x (ranges, ops, results)
    size_t h_slot = 0;
    cudaEvent_t done[2] = {};  // root: batch results copied to h_pin
    int64_t launches = 0;
    int flip = 0;
    std::mutex mu;
};

namespace {

bool exchanges(const Exec* e) { return e->own_comms || e->comm; }

void free_bufs(Exec* e) {
    for (DevCtx& d : e->dev) {
        DevGuard g(d.device);
        for (int p = 0; p < 2; ++p) {
            cudaFree(d.d_ranges[p]);
            cudaFree(d.d_ops[p]);
            cudaFree(d.acc_sum[p]);
            cudaFree(d.acc_ext[p]);
            cudaFree(d.d_res[p]);
            d.d_ranges[p] = nullptr;
            d.d_ops[p] = nullptr;
            d.acc_sum[p] = nullptr;
            d.acc_ext[p] = nullptr;
            d.d_res[p] = nullptr;
        }
        cudaFree(d.tmp_sum);
        cudaFree(d.tmp_ext);
        d.tmp_sum = nullptr;
        d.tmp_ext = nullptr;
    }
    cudaFreeHost(e->h_pin);
    e->h_pin = nullptr;
    e->cap = 0;
}

// wait for everything in flight on the executor's streams
int drain(Exec* e) {
    for (DevCtx& d : e->dev) {
        DevGuard g(d.device);
        if (d.cs) OLAP_CUDA_TRY(cudaStreamSynchronize(d.cs));
        if (d.ms) OLAP_CUDA_TRY(cudaStreamSynchronize(d.ms));
    }
    return OLAP_OK;
}

int ensure_cap(Exec* e, int64_t nq) {
    if (nq <= e->cap) return OLAP_OK;
    int rc = drain(e);
    if (rc) return rc;
    free_bufs(e);
    const int64_t cap = std::max<int64_t>(nq, 1024);
    for (DevCtx& d : e->dev) {
        DevGuard g(d.device);
        for (int p = 0; p < 2; ++p) {
            OLAP_CUDA_TRY(cudaMalloc(&d.d_ranges[p], sizeof(olap_range) * e->nd * cap));
            OLAP_CUDA_TRY(cudaMalloc(&d.d_ops[p], sizeof(int32_t) * cap));
            OLAP_CUDA_TRY(cudaMalloc(&d.acc_sum[p], sizeof(int64_t) * cap));
            OLAP_CUDA_TRY(cudaMalloc(&d.acc_ext[p], sizeof(int32_t) * 2 * cap));
            OLAP_CUDA_TRY(cudaMalloc(&d.d_res[p], sizeof(olap_result) * cap));
        }
        if (d.shards.size() > 1) {
            OLAP_CUDA_TRY(cudaMalloc(&d.tmp_sum, sizeof(int64_t) * cap));
            OLAP_CUDA_TRY(cudaMalloc(&d.tmp_ext, sizeof(int32_t) * 2 * cap));
        }
    }
    e->h_slot = (sizeof(olap_range) * e->nd + sizeof(int32_t) + sizeof(olap_result)) * cap;
    {
        DevGuard g(e->dev[0].device);
        OLAP_CUDA_TRY(cudaHostAlloc(reinterpret_cast<void**>(&e->h_pin), 2 * e->h_slot, cudaHostAllocPortable));
    }
    e->cap = cap;
    return OLAP_OK;
}

char* pin_ranges(Exec* e, int p) { return e->h_pin + p * e->h_slot; }
char* pin_ops(Exec* e, int p, int64_t cap) { return pin_ranges(e, p) + sizeof(olap_range) * e->nd * cap; }
char* pin_res(Exec* e, int p, int64_t cap) { return pin_ops(e, p, cap) + sizeof(int32_t) * cap; }

// Issue one batch (no host synchronisation).  Inputs: host (already in the pinned slot p) or
// device pointers on devices[0] (ready when `user` reaches this call).  Outputs: the pinned slot p
// (e->done[p] marks them complete) or d_results on devices[0] (`user` waits for them).
int issue(Exec* e, int p, int64_t nq, const olap_range* d_ranges_root, const int32_t* d_ops_root,
          olap_result* d_results_root, cudaStream_t user) {
    if (e->failed || (e->comm && e->comm->failed))
        return set_error(OLAP_E_NCCL, "the cube's communicator failed earlier; recreate it");
    const bool dev_in = d_ranges_root != nullptr;
    const size_t rb = sizeof(olap_range) * e->nd * nq, ob = sizeof(int32_t) * nq;
    DevCtx& root = e->dev[0];
    if (dev_in) {
        DevGuard g(root.device);
        OLAP_CUDA_TRY(cudaEventRecord(root.ev_in, user));
    }
    // ---- per device: inputs, shard partials, local combine (compute stream)
    for (DevCtx& d : e->dev) {
        DevGuard g(d.device);
        // slot p was last used two batches ago: its exchange / finalize must be done with it
        OLAP_CUDA_TRY(cudaStreamWaitEvent(d.cs, d.ev_free[p], 0));
        const olap_range* rng = d.d_ranges[p];
        const int32_t* ops = d.d_ops[p];
        if (dev_in) {
            OLAP_CUDA_TRY(cudaStreamWaitEvent(d.cs, root.ev_in, 0));
            if (&d == &root) {
                rng = d_ranges_root;
                ops = d_ops_root;
            } else {
                OLAP_CUDA_TRY(cudaMemcpyPeerAsync(d.d_ranges[p], d.device, d_ranges_root, root.device, rb, d.cs));
                OLAP_CUDA_TRY(cudaMemcpyPeerAsync(d.d_ops[p], d.device, d_ops_root, root.device, ob, d.cs));
            }
        } else {
            OLAP_CUDA_TRY(cudaMemcpyAsync(d.d_ranges[p], pin_ranges(e, p), rb, cudaMemcpyHostToDevice, d.cs));
            OLAP_CUDA_TRY(cudaMemcpyAsync(d.d_ops[p], pin_ops(e, p, e->cap), ob, cudaMemcpyHostToDevice, d.cs));
        }
        for (size_t j = 0; j < d.shards.size(); ++j) {
            int64_t* s = j == 0 ? d.acc_sum[p] : d.tmp_sum;
            int32_t* x = j == 0 ? d.acc_ext[p] : d.tmp_ext;
            int rc = olap_query_partials_device(d.shards[j], nq, rng, ops, s, x, d.cs);
            if (rc) return rc;
            if (j) {  // shards on one device fold in shard order (fixed: deterministic float sums)
                rc = olap_partials_combine_device(e->dtype, nq, d.tmp_sum, d.tmp_ext, d.acc_sum[p], d.acc_ext[p], d.cs);
                if (rc) return rc;
                ++e->launches;
            }
        }
        OLAP_CUDA_TRY(cudaEventRecord(d.ev_part[p], d.cs));
        OLAP_CUDA_TRY(cudaStreamWaitEvent(d.ms, d.ev_part[p], 0));
    }
    // ---- the exchange: one NCCL group, two reductions per device (exchange streams)
    if (exchanges(e)) {
        const NcclApi* api = e->api;
        const ncclDataType_t st = e->dtype == OLAP_FLOAT32 ? ncclFloat64 : ncclUint64;  // uint64: mod 2^64 (R7)
        OLAP_NCCL_TRY(api, api->GroupStart());
        for (DevCtx& d : e->dev) {
            DevGuard g(d.device);
            if (e->own_comms) {  // group: reduce to devices[0], which finalizes
                api->Reduce(d.acc_sum[p], d.acc_sum[p], (size_t)nq, st, ncclSum, 0, d.comm, d.ms);
                api->Reduce(d.acc_ext[p], d.acc_ext[p], (size_t)(2 * nq), ncclInt32, ncclMax, 0, d.comm, d.ms);
            } else {             // one rank per process: every rank finalizes every answer
                api->AllReduce(d.acc_sum[p], d.acc_sum[p], (size_t)nq, st, ncclSum, d.comm, d.ms);
                api->AllReduce(d.acc_ext[p], d.acc_ext[p], (size_t)(2 * nq), ncclInt32, ncclMax, d.comm, d.ms);
            }
        }
        ncclResult_t ge = api->GroupEnd();
        if (ge != ncclSuccess) {
            e->failed = true;
            return set_error(OLAP_E_NCCL, "ncclGroupEnd (partials exchange of %lld queries): %s", (long long)nq,
                             api->GetErrorString(ge));
        }
        for (DevCtx& d : e->dev) {
            bool failed = false;
            int rc = check_comm(api, d.comm, &failed);
            if (rc) {
                e->failed = true;
                if (e->comm) e->comm->failed = true;
                return rc;
            }
        }
    }
    // ---- finalize on the devices that hold the complete partials, results out
    for (size_t i = 0; i < e->dev.size(); ++i) {
        DevCtx& d = e->dev[i];
        DevGuard g(d.device);
        if (i == 0 || !e->own_comms) {
            const olap_range* rng = (dev_in && i == 0) ? d_ranges_root : d.d_ranges[p];
            const int32_t* ops = (dev_in && i == 0) ? d_ops_root : d.d_ops[p];
            olap_result* res = (d_results_root && i == 0) ? d_results_root : d.d_res[p];
            int rc = olap_finalize_device(e->nd, e->n, e->dtype, nq, rng, ops, d.acc_sum[p], d.acc_ext[p], res, d.ms);
            if (rc) return rc;  // (counted by olap_finalize_launches)
            if (i == 0 && !d_results_root)
                OLAP_CUDA_TRY(cudaMemcpyAsync(pin_res(e, p, e->cap), res, sizeof(olap_result) * nq,
                                              cudaMemcpyDeviceToHost, d.ms));
            if (i == 0) OLAP_CUDA_TRY(cudaEventRecord(e->done[p], d.ms));
        }
        OLAP_CUDA_TRY(cudaEventRecord(d.ev_free[p], d.ms));
    }
    if (d_results_root) {
        DevGuard g(root.device);
        OLAP_CUDA_TRY(cudaStreamWaitEvent(user, root.ev_free[p], 0));
    }
    return OLAP_OK;
}

int stage_in(Exec* e, int p, int64_t nq, const olap_range* ranges, const int32_t* ops) {
    std::memcpy(pin_ranges(e, p), ranges, sizeof(olap_range) * e->nd * nq);
    std::memcpy(pin_ops(e, p, e->cap), ops, sizeof(int32_t) * nq);
    return OLAP_OK;
}

int collect(Exec* e, int p, int64_t nq, olap_result* results) {
    DevGuard g(e->dev[0].device);
    OLAP_CUDA_TRY(cudaEventSynchronize(e->done[p]));
    std::memcpy(results, pin_res(e, p, e->cap), sizeof(olap_result) * nq);
    return OLAP_OK;
}

}  // namespace

int validate_queries(int nd, const int64_t* n, int64_t nq, const olap_range* ranges, const int32_t* ops) {
    for (int64_t q = 0; q < nq; ++q) {
        if (ops[q] < OLAP_SUM || ops[q] > OLAP_AVG)
            return set_error(OLAP_E_INVALID, "query %lld: unknown op %d", (long long)q, ops[q]);
        for (int k = 0; k < nd; ++k) {
            const olap_range r = ranges[q * nd + k];
            if (r.lo < 0 || r.hi >= n[k])
                return set_error(OLAP_E_RANGE, "query %lld dimension %d: range [%lld,%lld] outside [0,%lld)",
                                 (long long)q, k, (long long)r.lo, (long long)r.hi, (long long)n[k]);
        }
    }
    return OLAP_OK;
}

void exec_destroy(Exec* e) {
    if (!e) return;
    drain(e);
    free_bufs(e);
    for (DevCtx& d : e->dev) {
        DevGuard g(d.device);
        if (e->own_comms && d.comm && e->api) e->api->CommDestroy(d.comm);
        for (int p = 0; p < 2; ++p) {
            if (d.ev_part[p]) cudaEventDestroy(d.ev_part[p]);
            if (d.ev_free[p]) cudaEventDestroy(d.ev_free[p]);
        }
        if (d.ev_in) cudaEventDestroy(d.ev_in);
        if (d.cs) cudaStreamDestroy(d.cs);
        if (d.ms) cudaStreamDestroy(d.ms);
    }
    {
        DevGuard g(e->dev.empty() ? 0 : e->dev[0].device);
        for (int p = 0; p < 2; ++p)
            if (e->done[p]) cudaEventDestroy(e->done[p]);
    }
    delete e;
}

int exec_create(const ExecSpec& s, Exec** out) {
    Exec* e = new (std::nothrow) Exec();
    if (!e) return set_error(OLAP_E_NOMEM, "host allocation failed");
    e->nd = s.nd;
    e->dtype = s.dtype;
    for (int k = 0; k < s.nd; ++k) e->n[k] = s.n[k];
    e->comm = s.comm;
    e->own_comms = s.own_comms;
    if (s.own_comms || s.comm) {
        int rc = nccl_api(&e->api);
        if (rc) {
            delete e;
            return rc;
        }
    }
    e->dev.resize(s.devices.size());
    for (size_t i = 0; i < s.devices.size(); ++i) {
        DevCtx& d = e->dev[i];
        d.device = s.devices[i];
        for (int j = 0; j < s.spd; ++j) d.shards.push_back(s.shards[i * s.spd + j]);
        DevGuard g(d.device);
        if (!g.ok || cudaStreamCreateWithFlags(&d.cs, cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamCreateWithFlags(&d.ms, cudaStreamNonBlocking) != cudaSuccess ||
            cudaEventCreateWithFlags(&d.ev_in, cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&d.ev_part[0], cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&d.ev_part[1], cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&d.ev_free[0], cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&d.ev_free[1], cudaEventDisableTiming) != cudaSuccess) {
            cudaGetLastError();
            exec_destroy(e);
            return set_error(OLAP_E_CUDA, "stream/event setup on device %d failed", d.device);
        }
        if (i == 0 && (cudaEventCreateWithFlags(&e->done[0], cudaEventDisableTiming) != cudaSuccess ||
                       cudaEventCreateWithFlags(&e->done[1], cudaEventDisableTiming) != cudaSuccess)) {
            exec_destroy(e);
            return set_error(OLAP_E_CUDA, "event setup failed");
        }
        for (size_t k = 0; k < s.devices.size(); ++k)  // NVLink peer access for the input broadcast
            if (k != i && cudaDeviceEnablePeerAccess(s.devices[k], 0) != cudaSuccess) cudaGetLastError();
    }
    if (s.own_comms) {
        std::vector<ncclComm_t> comms(s.devices.size());
        ncclResult_t r = e->api->CommInitAll(comms.data(), (int)s.devices.size(), s.devices.data());
        if (r != ncclSuccess) {
            e->own_comms = false;
            exec_destroy(e);
            return set_error(OLAP_E_NCCL, "ncclCommInitAll over %d devices: %s", (int)s.devices.size(),
                             g_nccl.GetErrorString(r));
        }
        for (size_t i = 0; i < comms.size(); ++i) e->dev[i].comm = comms[i];
    } else if (s.comm) {
        e->dev[0].comm = s.comm->comm;
    }
    *out = e;
    return OLAP_OK;
}

int exec_query_batch(Exec* e, int64_t nq, const olap_range* ranges, const int32_t* ops, olap_result* results) {
    std::lock_guard<std::mutex> lk(e->mu);
    int rc = ensure_cap(e, nq);
    if (rc) return rc;
    // the pinned slot 0 may still feed an earlier batch's copies
    {
        DevGuard g(e->dev[0].device);
        OLAP_CUDA_TRY(cudaEventSynchronize(e->done[0]));
    }
    stage_in(e, 0, nq, ranges, ops);
    rc = issue(e, 0, nq, nullptr, nullptr, nullptr, nullptr);
    if (rc) return rc;
    return collect(e, 0, nq, results);
}

int exec_query_batch_device(Exec* e, int64_t nq, const olap_range* d_ranges, const int32_t* d_ops,
                            olap_result* d_results, cudaStream_t st) {
    std::lock_guard<std::mutex> lk(e->mu);
    int rc = ensure_cap(e, nq);
    if (rc) return rc;
    // alternate the slots so that consecutive device batches do not serialise on one slot
    const int p = (e->flip ^= 1);
    return issue(e, p, nq, d_ranges, d_ops, d_results, st);
}

int exec_query_stream(Exec* e, int64_t nq, const olap_range* ranges, const int32_t* ops, olap_result* results,
                      int64_t batch) {
    std::lock_guard<std::mutex> lk(e->mu);
    if (batch <= 0 || batch > nq) batch = nq;
    int rc = ensure_cap(e, batch);
    if (rc) return rc;
    {
        DevGuard g(e->dev[0].device);
        OLAP_CUDA_TRY(cudaEventSynchronize(e->done[0]));
        OLAP_CUDA_TRY(cudaEventSynchronize(e->done[1]));
    }
    const int64_t nb = (nq + batch - 1) / batch;
    for (int64_t b = 0; b < nb; ++b) {
        const int p = (int)(b & 1);
        const int64_t q0 = b * batch, n = std::min(batch, nq - q0);
        stage_in(e, p, n, ranges + q0 * e->nd, ops + q0);
        rc = issue(e, p, n, nullptr, nullptr, nullptr, nullptr);
        if (rc) return rc;
        if (b >= 1) {  // batch b is queued: collect b-1 while b reduces
            const int64_t pq0 = (b - 1) * batch;
            rc = collect(e, 1 - p, std::min(batch, nq - pq0), results + pq0);
            if (rc) return rc;
        }
    }
    const int64_t lq0 = (nb - 1) * batch;
    return collect(e, (int)((nb - 1) & 1), nq - lq0, results + lq0);
}

int64_t exec_launches(const Exec* e) { return e ? e->launches : 0; }

}  // namespace olap

// ------------------------------------------------------------------ C-ABI: communicators
using namespace olap;

extern "C" {

int olap_comm_unique_id(olap_comm_id* id) {
    clear_error();
    if (!id) return set_error(OLAP_E_INVALID, "olap_comm_unique_id: NULL argument");
    const NcclApi* api = nullptr;
    int rc = nccl_api(&api);
    if (rc) return rc;
    static_assert(sizeof(olap_comm_id) == sizeof(ncclUniqueId), "olap_comm_id mirrors ncclUniqueId");
    ncclUniqueId u;
    OLAP_NCCL_TRY(api, api->GetUniqueId(&u));
    std::memcpy(id, &u, sizeof(u));
    return OLAP_OK;
}

int olap_comm_init_rank(const olap_comm_id* id, int nranks, int rank, int device, olap_comm** out) {
    clear_error();
    if (!id || !out) return set_error(OLAP_E_INVALID, "olap_comm_init_rank: NULL argument");
    if (nranks < 1 || rank < 0 || rank >= nranks)
        return set_error(OLAP_E_INVALID, "rank %d of %d", rank, nranks);
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return set_error(OLAP_E_CUDA, "no CUDA device available (the library has no CPU fallback)");
    if (device < 0 || device >= ndev) return set_error(OLAP_E_INVALID, "device %d not in [0,%d)", device, ndev);
    const NcclApi* api = nullptr;
    int rc = nccl_api(&api);
    if (rc) return rc;
    DevGuard g(device);
    ncclUniqueId u;
    std::memcpy(&u, id, sizeof(u));
    ncclComm_t comm = nullptr;
    OLAP_NCCL_TRY(api, api->CommInitRank(&comm, nranks, u, rank));
    olap_comm* c = new (std::nothrow) olap_comm();
    if (!c) {
        api->CommDestroy(comm);
        return set_error(OLAP_E_NOMEM, "host allocation failed");
    }
    c->comm = comm;
    c->nranks = nranks;
    c->rank = rank;
    c->device = device;
    *out = c;
    return OLAP_OK;
}

int olap_comm_info(const olap_comm* c, int* nranks, int* rank, int* device) {
    clear_error();
    if (!c) return set_error(OLAP_E_INVALID, "communicator is NULL");
    if (nranks) *nranks = c->nranks;
    if (rank) *rank = c->rank;
    if (device) *device = c->device;
    return OLAP_OK;
}

int olap_comm_check(olap_comm* c) {
    clear_error();
    if (!c) return set_error(OLAP_E_INVALID, "communicator is NULL");
    if (c->failed) return set_error(OLAP_E_NCCL, "the communicator failed earlier");
    const NcclApi* api = nullptr;
    int rc = nccl_api(&api);
    if (rc) return rc;
    return check_comm(api, c->comm, &c->failed);
}

int olap_comm_destroy(olap_comm* c) {
    clear_error();
    if (!c) return OLAP_OK;
    const NcclApi* api = nullptr;
    if (nccl_api(&api) == OLAP_OK && c->comm) {
        DevGuard g(c->device);
        if (c->failed) api->CommAbort(c->comm);
        else api->CommDestroy(c->comm);
    }
    delete c;
    return OLAP_OK;
}

int olap_exchange_partials_device(olap_comm* c, int dtype, int64_t nq, int64_t* d_sum, int32_t* d_ext, void* stream) {
    clear_error();
    if (!c) return set_error(OLAP_E_INVALID, "communicator is NULL");
    if (dtype != OLAP_INT32 && dtype != OLAP_FLOAT32) return set_error(OLAP_E_INVALID, "bad dtype %d", dtype);
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq == 0) return OLAP_OK;
    if (!d_sum || !d_ext) return set_error(OLAP_E_INVALID, "NULL device buffer");
    if (c->failed) return set_error(OLAP_E_NCCL, "the communicator failed earlier");
    const NcclApi* api = nullptr;
    int rc = nccl_api(&api);
    if (rc) return rc;
    DevGuard g(c->device);
    cudaStream_t st = static_cast<cudaStream_t>(stream);
    const ncclDataType_t t = dtype == OLAP_FLOAT32 ? ncclFloat64 : ncclUint64;
    OLAP_NCCL_TRY(api, api->GroupStart());
    api->AllReduce(d_sum, d_sum, (size_t)nq, t, ncclSum, c->comm, st);
    api->AllReduce(d_ext, d_ext, (size_t)(2 * nq), ncclInt32, ncclMax, c->comm, st);
    OLAP_NCCL_TRY(api, api->GroupEnd());
    return check_comm(api, c->comm, &c->failed);
}

int olap_nccl_version(int* version) {
    clear_error();
    if (!version) return set_error(OLAP_E_INVALID, "NULL argument");
    const NcclApi* api = nullptr;
    int rc = nccl_api(&api);
    if (rc) return rc;
    *version = api->version;
    return OLAP_OK;
}

}  // extern "C"
