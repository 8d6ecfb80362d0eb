// Dev microbenchmark: throughput of reducing a shared-memory-resident 64 KB chunk many times
// (the inner loop a chunk-shared scan would run), SUM via F2F+DADD vs MIN via FMNMX.
#include <cstdio>
#include <cuda_runtime.h>
constexpr int C = 16384;  // cells per chunk
template <int OP>
__global__ void __launch_bounds__(256, 3) k(const float* __restrict__ g, int reps, double* out) {
    extern __shared__ float sm[];
    for (int i = threadIdx.x; i < C; i += 256) sm[i] = g[(size_t)blockIdx.x * C + i];
    __syncthreads();
    double s = 0.0;
    float mn = 1e30f, hi = 0.f, lo = 0.f;
    const float4* v = reinterpret_cast<const float4*>(sm);
    for (int r = 0; r < reps; ++r) {
        for (int i = threadIdx.x; i < C / 4; i += 256) {
            float4 x = v[i ^ (r & 7)];
            if (OP == 0) { s += (double)x.x; s += (double)x.y; s += (double)x.z; s += (double)x.w; }
            else if (OP == 2) {  // float-float accumulation (TwoSum), FMA pipe only
                float e[4] = {x.x, x.y, x.z, x.w};
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const float t = hi + e[q];
                    const float bp = t - hi;
                    lo += (hi - (t - bp)) + (e[q] - bp);
                    hi = t;
                }
            }
            else { mn = fminf(mn, fminf(fminf(x.x, x.y), fminf(x.z, x.w))); }
        }
    }
    if (OP == 2) s = (double)hi + (double)lo;
    if (OP == 0 || OP == 2) out[blockIdx.x * 256 + threadIdx.x] = s;
    else out[blockIdx.x * 256 + threadIdx.x] = mn;
}
int main() {
    const int blocks = 148 * 3, reps = 400;
    float* g; double* o;
    cudaMalloc(&g, sizeof(float) * (size_t)C * blocks);
    cudaMalloc(&o, sizeof(double) * blocks * 256);
    cudaMemset(g, 0, sizeof(float) * (size_t)C * blocks);
    cudaFuncSetAttribute(k<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, C * 4);
    cudaFuncSetAttribute(k<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, C * 4);
    cudaFuncSetAttribute(k<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, C * 4);
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int op = 0; op < 3; ++op) {
        for (int it = 0; it < 2; ++it) {
            cudaEventRecord(a);
            if (op == 0) k<0><<<blocks, 256, C * 4>>>(g, reps, o);
            else if (op == 1) k<1><<<blocks, 256, C * 4>>>(g, reps, o);
            else k<2><<<blocks, 256, C * 4>>>(g, reps, o);
            cudaEventRecord(b); cudaEventSynchronize(b);
            float ms; cudaEventElapsedTime(&ms, a, b);
            double bytes = (double)blocks * reps * C * 4;
            if (it) printf("%s: %.2f ms  %.1f TB/s of cells read from smem\n", op == 1 ? "MIN (FMNMX)" : (op == 2 ? "SUM (TwoSum f32)" : "SUM (F2F+DADD)"), ms, bytes / ms / 1e9);
        }
    }
    return 0;
}
