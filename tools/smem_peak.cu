// Shared-memory read bandwidth of one B200, measured (the roofline denominator of the tile-shared
// scan, DESIGN.md §6/§9).  One 1,024-thread CTA per SM (the tile kernel's shape) and, as a check,
// 2 x 512-thread CTAs per SM.  Each thread streams conflict-free ld.shared.v4 / .v2 / .b32 loads
// over a 96 KiB buffer and folds them with one LOP3 per word (XOR), so the shared-memory pipe, not
// the ALU, is the limit.  Reports bytes per SM clock (from clock64 inside the kernel, so it does not
// depend on the clock the run got) and TB/s over the whole GPU from CUDA-event time.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/smem_peak tools/smem_peak.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int kBufBytes = 96 * 1024;

template <int W>  // bytes per load: 16, 8, 4
__global__ void smem_read(int reps, unsigned* out, unsigned long long* cycles) {
    extern __shared__ __align__(16) unsigned char sm[];
    for (int i = threadIdx.x; i < kBufBytes / 4; i += blockDim.x) reinterpret_cast<unsigned*>(sm)[i] = i * 2654435761u;
    __syncthreads();
    const int n = kBufBytes / W;  // loads per sweep
    unsigned a0 = 0, a1 = 0, a2 = 0, a3 = 0;
    const unsigned long long c0 = clock64();
    for (int r = 0; r < reps; ++r) {
#pragma unroll 8
        for (int i = threadIdx.x; i < n; i += blockDim.x) {
            const int idx = i ^ (r & 1);  // defeat loop-invariant hoisting; stays conflict-free
            if (W == 16) {
                const uint4 v = reinterpret_cast<const uint4*>(sm)[idx];
                a0 ^= v.x; a1 ^= v.y; a2 ^= v.z; a3 ^= v.w;
            } else if (W == 8) {
                const uint2 v = reinterpret_cast<const uint2*>(sm)[idx];
                a0 ^= v.x; a1 ^= v.y;
            } else {
                a0 ^= reinterpret_cast<const unsigned*>(sm)[idx];
            }
        }
    }
    __syncthreads();
    const unsigned long long c1 = clock64();
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 ^ a1 ^ a2 ^ a3;
    if (threadIdx.x == 0) cycles[blockIdx.x] = c1 - c0;
}

template <int W>
void run(int sms, int cps, int threads, int reps) {
    const int blocks = sms * cps;
    unsigned* out;
    unsigned long long* cyc;
    cudaMalloc(&out, sizeof(unsigned) * blocks * threads);
    cudaMalloc(&cyc, sizeof(unsigned long long) * blocks);
    cudaFuncSetAttribute(smem_read<W>, cudaFuncAttributeMaxDynamicSharedMemorySize, kBufBytes);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    smem_read<W><<<blocks, threads, kBufBytes>>>(2, out, cyc);  // warm-up
    cudaEventRecord(a);
    smem_read<W><<<blocks, threads, kBufBytes>>>(reps, out, cyc);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, a, b);
    unsigned long long* h = new unsigned long long[blocks];
    cudaMemcpy(h, cyc, sizeof(unsigned long long) * blocks, cudaMemcpyDeviceToHost);
    double cmax = 0;
    for (int i = 0; i < blocks; ++i) cmax = h[i] > cmax ? h[i] : cmax;
    const double bytes_sm = (double)cps * reps * kBufBytes;  // per SM
    int clk_khz = 0;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    printf("ld.shared %2d B, %d CTA/SM x %4d thr: %6.1f B/clk/SM (clock64), %6.2f TB/s over %d SMs (event time %.3f ms)"
           "  -> %.2f TB/s at the %d MHz max clock\n",
           W, cps, threads, bytes_sm / cmax, bytes_sm * sms / (ms * 1e-3) / 1e12, sms, ms,
           bytes_sm / cmax * sms * clk_khz * 1e3 / 1e12, clk_khz / 1000);
    delete[] h;
    cudaFree(out);
    cudaFree(cyc);
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    const int reps = 4000;
    run<16>(sms, 1, 1024, reps);
    run<8>(sms, 1, 1024, reps);
    run<4>(sms, 1, 1024, reps);
    run<16>(sms, 2, 512, reps);
    run<16>(sms, 1, 1024, reps);  // repeat: steady clocks
    return 0;
}
