// common.cuh — internal helpers of the B200 OLAP library (not part of the C-ABI).
//
// Error reporting, fast 32-bit division by run-time constants, block-cyclic
// shard geometry (reading R3) and the dictionary hash.
// Everything here is product code; nothing is shared with oracle/.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <cstdarg>
#include <cstdio>
#include <string>

#include "olap.h"

#define OLAP_HD __host__ __device__ __forceinline__

namespace olap {

// ------------------------------------------------------------------ errors
int set_error(int status, const char* fmt, ...);
void clear_error();

#define OLAP_CUDA_TRY(expr)                                                                   \
    do {                                                                                      \
        cudaError_t e_ = (expr);                                                              \
        if (e_ != cudaSuccess)                                                                \
            return ::olap::set_error(e_ == cudaErrorMemoryAllocation ? OLAP_E_NOMEM : OLAP_E_CUDA, \
                                     "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(e_),  \
                                     __FILE__, __LINE__);                                     \
    } while (0)

// ------------------------------------------------------------------ fast division
// q = n / d for 0 <= n < 2^31 and 1 <= d < 2^31, branch-free (Granlund-Montgomery,
// 33-bit magic): l = ceil(log2 d), m = floor(2^32 (2^l - d) / d) + 1,
// q = (mulhi(n, m) + n) >> l   (no overflow: mulhi(n,m) + n < 2n < 2^32).
// Verified exhaustively for small d and randomly for large d by
// tests/test_host_logic.py (through olap_selftest_fastdiv).
struct FastDiv {
    uint32_t d, m, l;
};

inline FastDiv make_fastdiv(uint32_t d) {
    FastDiv f;
    f.d = d;
    uint32_t l = 0;
    while ((1ull << l) < d) ++l;  // ceil(log2 d)
    f.l = l;
    f.m = (uint32_t)(((1ull << 32) * ((1ull << l) - d)) / d + 1);
    return f;
}

OLAP_HD uint32_t fdiv(uint32_t n, const FastDiv& f) {
#ifdef __CUDA_ARCH__
    return (__umulhi(n, f.m) + n) >> f.l;
#else
    return (uint32_t)((((uint64_t)n * f.m) >> 32) + n) >> f.l;
#endif
}

// ------------------------------------------------------------------ shard geometry
// Block-cyclic dim-0 sharding: row r -> shard (r / b) % G, local row
// (r / (b*G))*b + r % b.  A global range [lo,hi] maps to ONE contiguous local
// range [L(f'), L(t')] where f' / t' are the first / last owned rows inside it.
OLAP_HD int64_t shard_rows(int64_t n0, int64_t G, int64_t g, int64_t b) {
    int64_t cyc = b * G, full = n0 / cyc, rem = n0 % cyc;
    int64_t extra = rem - g * b;
    extra = extra < 0 ? 0 : (extra > b ? b : extra);
    return full * b + extra;
}

OLAP_HD int64_t shard_local_of(int64_t r, int64_t G, int64_t b) { return (r / (b * G)) * b + r % b; }

OLAP_HD int64_t shard_global_of(int64_t lr, int64_t G, int64_t g, int64_t b) {
    return (lr / b) * (b * G) + g * b + lr % b;
}

// local [*llo,*lhi] of global [lo,hi] (lo <= hi, inside [0,n0)); returns false if no owned row
OLAP_HD bool shard_local_range(int64_t n0, int64_t G, int64_t g, int64_t b, int64_t lo, int64_t hi,
                               int64_t* llo, int64_t* lhi) {
    if (G == 1) {
        *llo = lo;
        *lhi = hi;
        return lo <= hi;
    }
    const int64_t cyc = b * G, own0 = g * b, own1 = g * b + b;  // owned offsets [own0, own1) in a cycle
    int64_t c = lo / cyc, off = lo % cyc, f;
    if (off < own0) f = c * cyc + own0;
    else if (off < own1) f = lo;
    else f = (c + 1) * cyc + own0;
    c = hi / cyc;
    off = hi % cyc;
    int64_t t;
    if (off >= own1) t = c * cyc + own1 - 1;
    else if (off >= own0) t = hi;
    else t = c * cyc - cyc + own1 - 1;  // previous cycle (may be negative)
    if (t > n0 - 1) t = n0 - 1;
    if (f > t || t < 0) return false;
    *llo = shard_local_of(f, G, b);
    *lhi = shard_local_of(t, G, b);
    return true;
}

// ------------------------------------------------------------------ dictionary hash
// Order-free over 4-byte words so a warp can hash a key in parallel:
//   h = fmix64( sum_j fmix64((j << 32 | w_j) + K1)  +  len * K2 )   (mod 2^64)
// where w_j is the little-endian word of bytes [4j, 4j+4) zero-padded.
OLAP_HD uint64_t fmix64(uint64_t k) {
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    k *= 0xc4ceb9fe1a85ec53ull;
    k ^= k >> 33;
    return k;
}
OLAP_HD uint64_t hash_word(uint32_t j, uint32_t w) {
    return fmix64((((uint64_t)j << 32) | w) + 0x9E3779B97F4A7C15ull);
}
OLAP_HD uint64_t hash_final(uint64_t sum, uint64_t len) { return fmix64(sum + len * 0xD6E8FEB86659FD93ull); }

inline uint64_t hash_bytes_host(const unsigned char* p, int64_t len) {
    uint64_t s = 0;
    for (int64_t j = 0; 4 * j < len; ++j) {
        uint32_t w = 0;
        for (int k = 0; k < 4 && 4 * j + k < len; ++k) w |= (uint32_t)p[4 * j + k] << (8 * k);
        s += hash_word((uint32_t)j, w);
    }
    return hash_final(s, (uint64_t)len);
}

constexpr uint64_t kEmptySlot = ~0ull;  // slot = (tag32 << 32) | id ; ids < 2^31

}  // namespace olap
