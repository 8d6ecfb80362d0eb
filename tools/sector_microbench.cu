// DRAM fetch granularity for isolated 32-B reads (C5's short runs): each thread reads one
// 32-B sector at a pseudo-random 256-B-aligned address of an 8 GiB buffer, with different
// load flavours.  Run under ncu (dram__bytes_read.sum per kernel) to see how many DRAM bytes
// one isolated sector costs.  Development aid, not part of the library.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint64_t mix(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}

template <int MODE>
__global__ void probe(const uint32_t* __restrict__ buf, uint64_t nlines, uint64_t n, uint32_t* out) {
    uint32_t acc = 0;
    uint64_t pol = 0;
    if (MODE == 6) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t* p = buf + (mix(i) % nlines) * 64;  // 256-B lines, read the first 32 B
        uint32_t r[8];
        if (MODE == 0) {
            asm volatile("ld.global.nc.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                         : "l"(p));
        } else if (MODE == 1) {
            asm volatile("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                         : "l"(p));
        } else if (MODE == 2) {
            asm volatile("ld.global.cg.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                         : "l"(p));
        } else if (MODE == 3) {
            asm volatile("ld.global.cs.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                         : "l"(p));
        } else if (MODE == 4) {  // one 16-B load only
            asm volatile("ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "l"(p));
            r[4] = r[5] = r[6] = r[7] = 0;
        } else if (MODE == 5) {  // 4-B load
            asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(r[0]) : "l"(p));
            r[1] = r[2] = r[3] = r[4] = r[5] = r[6] = r[7] = 0;
        } else if (MODE == 6) {
            asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7])
                         : "l"(p), "l"(pol));
        } else if (MODE == 7) {  // volatile (ld.volatile.global): no L1, strong ordering off
            asm volatile("ld.volatile.global.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]) : "l"(p));
            asm volatile("ld.volatile.global.v4.u32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]) : "l"(p + 4));
        }
#pragma unroll
        for (int k = 0; k < 8; ++k) acc += r[k];
    }
    if (acc == 0x12345678u) out[0] = acc;
}

int main(int argc, char** argv) {
    const uint64_t bytes = 8ull << 30, nlines = bytes / 256, n = 1ull << 26;  // 2^26 sectors = 2 GiB useful
    uint32_t* buf;
    uint32_t* out;
    if (cudaMalloc(&buf, bytes) != cudaSuccess || cudaMalloc(&out, 4) != cudaSuccess) return 1;
    cudaMemset(buf, 1, bytes);
    int lim = argc > 1 ? atoi(argv[1]) : 0;
    if (lim) cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, lim);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    auto run = [&](auto kern, const char* name) {
        kern<<<148 * 8, 256>>>(buf, nlines, n, out);
        cudaEventRecord(a);
        kern<<<148 * 8, 256>>>(buf, nlines, n, out);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        printf("%-40s %8.3f ms  %7.1f GB/s useful (32 B per read)\n", name, ms, n * 32.0 / ms / 1e6);
    };
    run(probe<0>, "nc.v8 (LDG.256, L1 allocate)");
    run(probe<1>, "nc.L1::no_allocate.v8");
    run(probe<2>, "cg.v8 (L2 only)");
    run(probe<3>, "cs.v8 (streaming)");
    run(probe<4>, "nc.v4 (16 B)");
    run(probe<5>, "nc.u32 (4 B)");
    run(probe<6>, "nc.no_allocate + L2 evict_first policy");
    run(probe<7>, "volatile 2 x v4");
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
