// dict.cu — text-to-integer translation with one dictionary per text column
// (§III-F).  The paper searched each dictionary linearly on one
// CPU thread (Eq. 17: 13.8 ns per entry).  Here a dictionary is a
// sorted arena of its distinct keys (id = rank, reading R11) plus an open-addressing
// hash table of (tag32, id) slots; translation is one warp per key on the GPU:
// lane-parallel hash, 32-slot parallel probe with ballot, cooperative byte compare.
#include <algorithm>
#include <cstring>
#include <new>
#include <numeric>
#include <vector>

#include "common.cuh"

namespace olap {

constexpr int kMaxDicts = 32;

struct DictDev {
    const unsigned char* arena;
    const int64_t* offs;
    const unsigned long long* table;
    unsigned long long mask;
    int64_t D;
};

struct DictSet {
    DictDev d[kMaxDicts];
};

// key i of the query arena vs member `id`: <0, 0, >0 (memcmp order, shorter prefix first)
__device__ int warp_compare(const unsigned char* __restrict__ kp, int64_t klen, const DictDev& dd, int64_t id,
                            int lane) {
    const int64_t ma = dd.offs[id], mlen = dd.offs[id + 1] - ma;
    const unsigned char* mp = dd.arena + ma;
    const int64_t m = klen < mlen ? klen : mlen;
    for (int64_t j0 = 0; j0 < m; j0 += 32) {
        const int64_t j = j0 + lane;
        const unsigned char a = j < m ? kp[j] : 0, b = j < m ? mp[j] : 0;
        const unsigned diff = __ballot_sync(0xffffffffu, a != b);
        if (diff) {
            const int l = __ffs(diff) - 1;
            const int av = __shfl_sync(0xffffffffu, (int)a, l), bv = __shfl_sync(0xffffffffu, (int)b, l);
            return av - bv;
        }
    }
    return klen < mlen ? -1 : (klen > mlen ? 1 : 0);
}

// id of the key [kp, kp+len) in dd, or -1 (warp-cooperative: hash, 32-slot probe, compare)
__device__ int32_t translate_one(const DictDev& dd, const unsigned char* __restrict__ kp, int64_t len, int lane) {
    unsigned long long s = 0ull;
    for (int64_t j = lane; 4 * j < len; j += 32) {
        uint32_t wd = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k)
            if (4 * j + k < len) wd |= (uint32_t)kp[4 * j + k] << (8 * k);
        s += hash_word((uint32_t)j, wd);
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const unsigned long long h = hash_final(s, (unsigned long long)len);
    const uint32_t tag = (uint32_t)(h >> 32);
    unsigned long long pos = h & dd.mask;
    if (dd.D <= 0) return -1;
    for (;;) {
        const unsigned long long slot = dd.table[(pos + lane) & dd.mask];
        const bool empty = slot == kEmptySlot;
        const bool cand = !empty && (uint32_t)(slot >> 32) == tag;
        const unsigned me = __ballot_sync(0xffffffffu, empty);
        unsigned mc = __ballot_sync(0xffffffffu, cand);
        if (me) mc &= (me & (0u - me)) - 1u;  // only candidates before the first empty slot
        while (mc) {
            const int l = __ffs(mc) - 1;
            mc &= mc - 1;
            const int64_t id = (int64_t)(uint32_t)__shfl_sync(0xffffffffu, (unsigned long long)slot, l);
            if (warp_compare(kp, len, dd, id, lane) == 0) return (int32_t)id;
        }
        if (me) return -1;
        pos += 32;
    }
}

// number of members < key (upper = 0) or <= key (upper = 1): warp-cooperative binary search
__device__ int64_t bound_one(const DictDev& dd, const unsigned char* __restrict__ kp, int64_t len, int upper,
                             int lane) {
    int64_t lo = 0, hi = dd.D;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        const int c = warp_compare(kp, len, dd, mid, lane);  // key vs member(mid)
        if (c > 0 || (upper && c == 0)) lo = mid + 1;
        else hi = mid;
    }
    return lo;
}

__global__ void translate_kernel(DictSet ds, int ndicts, const int32_t* __restrict__ dict_of_key,
                                 const unsigned char* __restrict__ bytes, const int64_t* __restrict__ offs, int64_t n,
                                 int32_t* __restrict__ ids, unsigned long long* nmiss) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t key = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; key < n; key += warps) {
        const int di = dict_of_key ? dict_of_key[key] : 0;
        int32_t result = -1;
        if (di >= 0 && di < ndicts) {
            const int64_t a = offs[key];
            result = translate_one(ds.d[di], bytes + a, offs[key + 1] - a, lane);
        }
        if (lane == 0) {
            ids[key] = result;
            if (result < 0 && nmiss) atomicAdd(nmiss, 1ull);
        }
    }
}

__global__ void bound_kernel(DictDev dd, const unsigned char* __restrict__ bytes, const int64_t* __restrict__ offs,
                             int64_t n, int upper, int32_t* __restrict__ out) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t key = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; key < n; key += warps) {
        const int64_t a = offs[key];
        const int64_t r = bound_one(dd, bytes + a, offs[key + 1] - a, upper, lane);
        if (lane == 0) out[key] = (int32_t)r;
    }
}

struct Ext8 {
    int64_t n[8];
};

// One warp per (query, dimension) condition: text -> Eq. 1 range (readings R11, R13).
__global__ void text_ranges_kernel(DictSet ds, int ndims, Ext8 ext, int64_t nq, const int32_t* __restrict__ kinds,
                                   const int64_t* __restrict__ first_key, const olap_range* __restrict__ rin,
                                   const unsigned char* __restrict__ bytes, const int64_t* __restrict__ offs,
                                   int64_t nkeys, olap_range* __restrict__ rout, unsigned long long* nmiss) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const int64_t nc = nq * ndims;
    for (int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < nc; c += warps) {
        const int d = (int)(c % ndims);
        const int32_t kind = kinds[c];
        olap_range r;
        r.lo = -1;  // invalid unless set below: the query is then flagged / rejected
        r.hi = -1;
        bool miss = false;
        if (kind == OLAP_COND_ALL) {
            r.lo = 0;
            r.hi = ext.n[d] - 1;
        } else if (kind == OLAP_COND_IDS) {
            if (rin) r = rin[c];
        } else if (kind == OLAP_COND_EQ || kind == OLAP_COND_RANGE) {
            const int64_t k = first_key[c];
            const int64_t need = kind == OLAP_COND_EQ ? 1 : 2;
            if (k >= 0 && k + need <= nkeys && ds.d[d].table) {
                const DictDev& dd = ds.d[d];
                const int64_t a = offs[k];
                if (kind == OLAP_COND_EQ) {
                    const int32_t id = translate_one(dd, bytes + a, offs[k + 1] - a, lane);
                    if (id >= 0) {
                        r.lo = id;
                        r.hi = id;
                    } else {
                        r.lo = 1;  // empty box
                        r.hi = 0;
                        miss = true;
                    }
                } else {
                    const int64_t b = offs[k + 1];
                    r.lo = bound_one(dd, bytes + a, b - a, 0, lane);
                    r.hi = bound_one(dd, bytes + b, offs[k + 2] - b, 1, lane) - 1;
                }
            }
        }
        if (lane == 0) {
            rout[c] = r;
            if (miss && nmiss) atomicAdd(nmiss, 1ull);
        }
    }
}

}  // namespace olap

using namespace olap;

struct olap_dict {
    int device = 0;
    int64_t D = 0;
    std::vector<unsigned char> arena;
    std::vector<int64_t> offs;
    unsigned char* d_arena = nullptr;
    int64_t* d_offs = nullptr;
    unsigned long long* d_table = nullptr;
    unsigned long long mask = 0;
};

namespace {

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

int check_keys(const char* bytes, const int64_t* offsets, int64_t n) {
    if (n < 0) return set_error(OLAP_E_INVALID, "n < 0");
    if (n > 0 && (!offsets || (!bytes && offsets[n] > offsets[0])))
        return set_error(OLAP_E_INVALID, "NULL key buffer");
    for (int64_t i = 0; i < n; ++i)
        if (offsets[i] < 0 || offsets[i + 1] < offsets[i])
            return set_error(OLAP_E_INVALID, "offsets not non-decreasing at %lld", (long long)i);
    return OLAP_OK;
}

DictDev dev_view(const olap_dict* d) {
    DictDev v;
    v.arena = d->d_arena;
    v.offs = d->d_offs;
    v.table = d->d_table;
    v.mask = d->mask;
    v.D = d->D;
    return v;
}

int grid_for(int64_t n) { return (int)std::max<int64_t>(1, std::min<int64_t>((n + 7) / 8, 148 * 32)); }

}  // namespace

extern "C" {

int olap_dict_build(const char* bytes, const int64_t* offsets, int64_t n, int device, olap_dict** out) {
    clear_error();
    if (!out) return set_error(OLAP_E_INVALID, "out is NULL");
    int rc = check_keys(bytes, offsets, n);
    if (rc) return rc;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0)
        return set_error(OLAP_E_CUDA, "no CUDA device available (the library has no CPU fallback)");
    if (device < 0 || device >= ndev) return set_error(OLAP_E_INVALID, "device %d not in [0,%d)", device, ndev);
    const unsigned char* ub = reinterpret_cast<const unsigned char*>(bytes);
    // sort key indices in memcmp order (shorter prefix first), then unique -> ids = ranks
    std::vector<int64_t> idx(n);
    std::iota(idx.begin(), idx.end(), 0);
    auto less = [&](int64_t x, int64_t y) {
        const int64_t lx = offsets[x + 1] - offsets[x], ly = offsets[y + 1] - offsets[y];
        const int c = std::memcmp(ub + offsets[x], ub + offsets[y], (size_t)std::min(lx, ly));
        return c != 0 ? c < 0 : lx < ly;
    };
    std::sort(idx.begin(), idx.end(), less);
    olap_dict* d = new (std::nothrow) olap_dict();
    if (!d) return set_error(OLAP_E_NOMEM, "host allocation failed");
    d->device = device;
    d->offs.push_back(0);
    for (int64_t k = 0; k < n; ++k) {
        const int64_t i = idx[k];
        if (k > 0 && !less(idx[k - 1], i)) continue;  // duplicate
        d->arena.insert(d->arena.end(), ub + offsets[i], ub + offsets[i + 1]);
        d->offs.push_back((int64_t)d->arena.size());
    }
    d->D = (int64_t)d->offs.size() - 1;
    if (d->D >= (1ll << 31) - 1) {
        delete d;
        return set_error(OLAP_E_UNSUPPORTED, "more than 2^31-2 distinct keys");
    }
    uint64_t cap = 64;
    while (cap < (uint64_t)(2 * d->D)) cap <<= 1;
    d->mask = cap - 1;
    std::vector<unsigned long long> table(cap, kEmptySlot);
    for (int64_t id = 0; id < d->D; ++id) {
        const uint64_t h = hash_bytes_host(d->arena.data() + d->offs[id], d->offs[id + 1] - d->offs[id]);
        uint64_t pos = h & d->mask;
        while (table[pos] != kEmptySlot) pos = (pos + 1) & d->mask;
        table[pos] = ((h >> 32) << 32) | (uint64_t)id;
    }
    DevGuard g(device);
    cudaError_t e = cudaSuccess;
    const size_t abytes = std::max<size_t>(d->arena.size(), 1);
    if ((e = cudaMalloc(&d->d_arena, abytes)) != cudaSuccess ||
        (e = cudaMalloc(&d->d_offs, sizeof(int64_t) * d->offs.size())) != cudaSuccess ||
        (e = cudaMalloc(&d->d_table, sizeof(unsigned long long) * cap)) != cudaSuccess ||
        (!d->arena.empty() &&
         (e = cudaMemcpy(d->d_arena, d->arena.data(), d->arena.size(), cudaMemcpyHostToDevice)) != cudaSuccess) ||
        (e = cudaMemcpy(d->d_offs, d->offs.data(), sizeof(int64_t) * d->offs.size(), cudaMemcpyHostToDevice)) !=
            cudaSuccess ||
        (e = cudaMemcpy(d->d_table, table.data(), sizeof(unsigned long long) * cap, cudaMemcpyHostToDevice)) !=
            cudaSuccess) {
        rc = set_error(e == cudaErrorMemoryAllocation ? OLAP_E_NOMEM : OLAP_E_CUDA, "dictionary upload: %s",
                       cudaGetErrorString(e));
        cudaGetLastError();
        olap_dict_destroy(d);
        return rc;
    }
    *out = d;
    return OLAP_OK;
}

int olap_dict_size(const olap_dict* d, int64_t* n_distinct) {
    clear_error();
    if (!d || !n_distinct) return set_error(OLAP_E_INVALID, "NULL argument");
    *n_distinct = d->D;
    return OLAP_OK;
}

int olap_dict_translate_device(const olap_dict* const* dicts, int ndicts, const int32_t* d_dict_of_key,
                               const char* d_bytes, const int64_t* d_offsets, int64_t n, int32_t* d_ids_out,
                               int64_t* d_n_missing, void* stream) {
    clear_error();
    if (!dicts || ndicts < 1 || ndicts > kMaxDicts) return set_error(OLAP_E_INVALID, "ndicts must be in [1,32]");
    if (n < 0) return set_error(OLAP_E_INVALID, "n < 0");
    if (n == 0) return OLAP_OK;
    if (!d_offsets || !d_ids_out) return set_error(OLAP_E_INVALID, "NULL device buffer");
    DictSet ds;
    std::memset(&ds, 0, sizeof(ds));
    for (int i = 0; i < ndicts; ++i) {
        if (!dicts[i]) return set_error(OLAP_E_INVALID, "dicts[%d] is NULL", i);
        if (dicts[i]->device != dicts[0]->device) return set_error(OLAP_E_INVALID, "dictionaries on different devices");
        ds.d[i] = dev_view(dicts[i]);
    }
    DevGuard g(dicts[0]->device);
    translate_kernel<<<grid_for(n), 256, 0, static_cast<cudaStream_t>(stream)>>>(
        ds, ndicts, d_dict_of_key, reinterpret_cast<const unsigned char*>(d_bytes), d_offsets, n, d_ids_out,
        reinterpret_cast<unsigned long long*>(d_n_missing));
    OLAP_CUDA_TRY(cudaGetLastError());
    return OLAP_OK;
}

int olap_dict_translate(const olap_dict* const* dicts, int ndicts, const int32_t* dict_of_key, const char* bytes,
                        const int64_t* offsets, int64_t n, int32_t* ids_out, int64_t* n_missing) {
    clear_error();
    if (!dicts || ndicts < 1 || ndicts > kMaxDicts || !dicts[0])
        return set_error(OLAP_E_INVALID, "ndicts must be in [1,32]");
    int rc = check_keys(bytes, offsets, n);
    if (rc) return rc;
    if (n == 0) {
        if (n_missing) *n_missing = 0;
        return OLAP_OK;
    }
    if (!ids_out) return set_error(OLAP_E_INVALID, "ids_out is NULL");
    DevGuard g(dicts[0]->device);
    cudaStream_t st = cudaStreamPerThread;
    const int64_t base = offsets[0], nbytes = offsets[n] - base;
    std::vector<int64_t> offs(offsets, offsets + n + 1);
    for (auto& o : offs) o -= base;
    char* d_bytes = nullptr;
    int64_t* d_offs = nullptr;
    int32_t* d_dk = nullptr;
    int32_t* d_ids = nullptr;
    int64_t* d_miss = nullptr;
    OLAP_CUDA_TRY(cudaMallocAsync(&d_bytes, std::max<int64_t>(nbytes, 1), st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_offs, sizeof(int64_t) * (n + 1), st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_ids, sizeof(int32_t) * n, st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_miss, sizeof(int64_t), st));
    if (dict_of_key) OLAP_CUDA_TRY(cudaMallocAsync(&d_dk, sizeof(int32_t) * n, st));
    if (nbytes) OLAP_CUDA_TRY(cudaMemcpyAsync(d_bytes, bytes + base, nbytes, cudaMemcpyHostToDevice, st));
    OLAP_CUDA_TRY(cudaMemcpyAsync(d_offs, offs.data(), sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, st));
    if (dict_of_key)
        OLAP_CUDA_TRY(cudaMemcpyAsync(d_dk, dict_of_key, sizeof(int32_t) * n, cudaMemcpyHostToDevice, st));
    OLAP_CUDA_TRY(cudaMemsetAsync(d_miss, 0, sizeof(int64_t), st));
    rc = olap_dict_translate_device(dicts, ndicts, d_dk, d_bytes, d_offs, n, d_ids, d_miss, st);
    int64_t miss = 0;
    if (rc == OLAP_OK) {
        OLAP_CUDA_TRY(cudaMemcpyAsync(ids_out, d_ids, sizeof(int32_t) * n, cudaMemcpyDeviceToHost, st));
        OLAP_CUDA_TRY(cudaMemcpyAsync(&miss, d_miss, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    }
    cudaFreeAsync(d_bytes, st);
    cudaFreeAsync(d_offs, st);
    cudaFreeAsync(d_ids, st);
    cudaFreeAsync(d_miss, st);
    if (d_dk) cudaFreeAsync(d_dk, st);
    OLAP_CUDA_TRY(cudaStreamSynchronize(st));
    if (rc) return rc;
    if (n_missing) *n_missing = miss;
    return OLAP_OK;
}

int olap_dict_bound(const olap_dict* d, const char* bytes, const int64_t* offsets, int64_t n, int upper,
                    int32_t* out) {
    clear_error();
    if (!d) return set_error(OLAP_E_INVALID, "dict is NULL");
    int rc = check_keys(bytes, offsets, n);
    if (rc) return rc;
    if (n == 0) return OLAP_OK;
    if (!out) return set_error(OLAP_E_INVALID, "out is NULL");
    DevGuard g(d->device);
    cudaStream_t st = cudaStreamPerThread;
    const int64_t base = offsets[0], nbytes = offsets[n] - base;
    std::vector<int64_t> offs(offsets, offsets + n + 1);
    for (auto& o : offs) o -= base;
    char* d_bytes = nullptr;
    int64_t* d_offs = nullptr;
    int32_t* d_out = nullptr;
    OLAP_CUDA_TRY(cudaMallocAsync(&d_bytes, std::max<int64_t>(nbytes, 1), st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_offs, sizeof(int64_t) * (n + 1), st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_out, sizeof(int32_t) * n, st));
    if (nbytes) OLAP_CUDA_TRY(cudaMemcpyAsync(d_bytes, bytes + base, nbytes, cudaMemcpyHostToDevice, st));
    OLAP_CUDA_TRY(cudaMemcpyAsync(d_offs, offs.data(), sizeof(int64_t) * (n + 1), cudaMemcpyHostToDevice, st));
    bound_kernel<<<grid_for(n), 256, 0, st>>>(dev_view(d), reinterpret_cast<const unsigned char*>(d_bytes), d_offs, n,
                                              upper ? 1 : 0, d_out);
    OLAP_CUDA_TRY(cudaGetLastError());
    OLAP_CUDA_TRY(cudaMemcpyAsync(out, d_out, sizeof(int32_t) * n, cudaMemcpyDeviceToHost, st));
    cudaFreeAsync(d_bytes, st);
    cudaFreeAsync(d_offs, st);
    cudaFreeAsync(d_out, st);
    OLAP_CUDA_TRY(cudaStreamSynchronize(st));
    return OLAP_OK;
}

int olap_text_ranges_device(const olap_dict* const* dicts, int ndims, const int64_t* extents, int64_t nq,
                            const int32_t* d_kinds, const int64_t* d_first_key, const olap_range* d_ranges_in,
                            const char* d_bytes, const int64_t* d_offsets, int64_t nkeys, olap_range* d_ranges_out,
                            int64_t* d_n_missing, void* stream) {
    clear_error();
    if (!dicts || ndims < 1 || ndims > 8 || !extents) return set_error(OLAP_E_INVALID, "bad dicts/ndims/extents");
    if (nq < 0 || nkeys < 0) return set_error(OLAP_E_INVALID, "nq < 0 or nkeys < 0");
    if (nq == 0) return OLAP_OK;
    if (!d_kinds || !d_ranges_out || (nkeys > 0 && (!d_offsets || !d_first_key)))
        return set_error(OLAP_E_INVALID, "NULL device buffer");
    DictSet ds;
    std::memset(&ds, 0, sizeof(ds));
    int dev = -1;
    for (int i = 0; i < ndims; ++i) {
        if (!dicts[i]) continue;
        if (dev >= 0 && dicts[i]->device != dev) return set_error(OLAP_E_INVALID, "dictionaries on different devices");
        dev = dicts[i]->device;
        ds.d[i] = dev_view(dicts[i]);
    }
    Ext8 e;
    std::memset(&e, 0, sizeof(e));
    for (int i = 0; i < ndims; ++i) e.n[i] = extents[i];
    DevGuard g(dev >= 0 ? dev : 0);
    text_ranges_kernel<<<grid_for(nq * ndims), 256, 0, static_cast<cudaStream_t>(stream)>>>(
        ds, ndims, e, nq, d_kinds, d_first_key, d_ranges_in, reinterpret_cast<const unsigned char*>(d_bytes), d_offsets,
        nkeys, d_ranges_out, reinterpret_cast<unsigned long long*>(d_n_missing));
    OLAP_CUDA_TRY(cudaGetLastError());
    return OLAP_OK;
}

int olap_text_ranges(const olap_dict* const* dicts, int ndims, const int64_t* extents, int64_t nq, const int32_t* kinds,
                     const olap_range* ranges_in, const char* bytes, const int64_t* offsets, int64_t nkeys,
                     olap_range* ranges_out, int64_t* n_missing) {
    clear_error();
    if (!dicts || ndims < 1 || ndims > 8 || !extents) return set_error(OLAP_E_INVALID, "bad dicts/ndims/extents");
    if (nq < 0) return set_error(OLAP_E_INVALID, "nq < 0");
    if (nq > 0 && (!kinds || !ranges_out)) return set_error(OLAP_E_INVALID, "NULL buffer");
    int rc = check_keys(bytes, offsets, nkeys);
    if (rc) return rc;
    // first key of every condition; validate kinds, dictionaries and extents
    std::vector<int64_t> first((size_t)(nq * ndims));
    int64_t k = 0;
    bool any_ids = false;
    int dev = -1;
    for (int64_t c = 0; c < nq * ndims; ++c) {
        const int d = (int)(c % ndims);
        const int32_t kind = kinds[c];
        first[c] = k;
        if (kind == OLAP_COND_EQ || kind == OLAP_COND_RANGE) {
            if (!dicts[d]) return set_error(OLAP_E_INVALID, "query %lld dimension %d: text condition on a dimension "
                                            "without a dictionary", (long long)(c / ndims), d);
            if (dicts[d]->D != extents[d])
                return set_error(OLAP_E_INVALID, "dimension %d: extent %lld != dictionary size %lld", d,
                                 (long long)extents[d], (long long)dicts[d]->D);
            dev = dicts[d]->device;
            k += kind == OLAP_COND_EQ ? 1 : 2;
        } else if (kind == OLAP_COND_IDS) {
            any_ids = true;
        } else if (kind != OLAP_COND_ALL) {
            return set_error(OLAP_E_INVALID, "query %lld dimension %d: unknown condition kind %d",
                             (long long)(c / ndims), d, kind);
        }
    }
    if (k != nkeys) return set_error(OLAP_E_INVALID, "conditions consume %lld keys, %lld given", (long long)k,
                                     (long long)nkeys);
    if (any_ids && !ranges_in) return set_error(OLAP_E_INVALID, "OLAP_COND_IDS needs ranges_in");
    if (nq == 0) {
        if (n_missing) *n_missing = 0;
        return OLAP_OK;
    }
    if (dev < 0)
        for (int i = 0; i < ndims; ++i)
            if (dicts[i]) dev = dicts[i]->device;
    DevGuard g(dev >= 0 ? dev : 0);
    cudaStream_t st = cudaStreamPerThread;
    const int64_t nc = nq * ndims;
    const int64_t base = nkeys ? offsets[0] : 0, nbytes = nkeys ? offsets[nkeys] - base : 0;
    std::vector<int64_t> offs;
    if (nkeys) {
        offs.assign(offsets, offsets + nkeys + 1);
        for (auto& o : offs) o -= base;
    }
    char* d_bytes = nullptr;
    int64_t *d_offs = nullptr, *d_first = nullptr, *d_miss = nullptr;
    int32_t* d_kinds = nullptr;
    olap_range *d_in = nullptr, *d_out = nullptr;
    OLAP_CUDA_TRY(cudaMallocAsync(&d_bytes, std::max<int64_t>(nbytes, 1), st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_offs, sizeof(int64_t) * (nkeys + 1), st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_first, sizeof(int64_t) * nc, st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_miss, sizeof(int64_t), st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_kinds, sizeof(int32_t) * nc, st));
    OLAP_CUDA_TRY(cudaMallocAsync(&d_out, sizeof(olap_range) * nc, st));
    if (any_ids) OLAP_CUDA_TRY(cudaMallocAsync(&d_in, sizeof(olap_range) * nc, st));
    if (nbytes) OLAP_CUDA_TRY(cudaMemcpyAsync(d_bytes, bytes + base, nbytes, cudaMemcpyHostToDevice, st));
    if (nkeys)
        OLAP_CUDA_TRY(cudaMemcpyAsync(d_offs, offs.data(), sizeof(int64_t) * (nkeys + 1), cudaMemcpyHostToDevice, st));
    OLAP_CUDA_TRY(cudaMemcpyAsync(d_first, first.data(), sizeof(int64_t) * nc, cudaMemcpyHostToDevice, st));
    OLAP_CUDA_TRY(cudaMemcpyAsync(d_kinds, kinds, sizeof(int32_t) * nc, cudaMemcpyHostToDevice, st));
    if (any_ids) OLAP_CUDA_TRY(cudaMemcpyAsync(d_in, ranges_in, sizeof(olap_range) * nc, cudaMemcpyHostToDevice, st));
    OLAP_CUDA_TRY(cudaMemsetAsync(d_miss, 0, sizeof(int64_t), st));
    rc = olap_text_ranges_device(dicts, ndims, extents, nq, d_kinds, d_first, d_in, d_bytes, d_offs, nkeys, d_out,
                                 d_miss, st);
    int64_t miss = 0;
    if (rc == OLAP_OK) {
        OLAP_CUDA_TRY(cudaMemcpyAsync(ranges_out, d_out, sizeof(olap_range) * nc, cudaMemcpyDeviceToHost, st));
        OLAP_CUDA_TRY(cudaMemcpyAsync(&miss, d_miss, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    }
    cudaFreeAsync(d_bytes, st);
    cudaFreeAsync(d_offs, st);
    cudaFreeAsync(d_first, st);
    cudaFreeAsync(d_miss, st);
    cudaFreeAsync(d_kinds, st);
    cudaFreeAsync(d_out, st);
    if (d_in) cudaFreeAsync(d_in, st);
    OLAP_CUDA_TRY(cudaStreamSynchronize(st));
    if (rc) return rc;
    if (n_missing) *n_missing = miss;
    return OLAP_OK;
}

int olap_dict_lookup(const olap_dict* d, int32_t id, const char** bytes, int64_t* len) {
    clear_error();
    if (!d || !bytes || !len) return set_error(OLAP_E_INVALID, "NULL argument");
    if (id < 0 || id >= d->D) return set_error(OLAP_E_RANGE, "id %d not in [0,%lld)", id, (long long)d->D);
    *bytes = reinterpret_cast<const char*>(d->arena.data() + d->offs[id]);
    *len = d->offs[id + 1] - d->offs[id];
    return OLAP_OK;
}

int olap_dict_destroy(olap_dict* d) {
    clear_error();
    if (!d) return OLAP_OK;
    DevGuard g(d->device);
    cudaFree(d->d_arena);
    cudaFree(d->d_offs);
    cudaFree(d->d_table);
    delete d;
    return OLAP_OK;
}

}  // extern "C"
