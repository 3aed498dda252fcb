// Probe: issue cost (SM cycles per warp-instruction) of the load paths a
// decode can use for the x segment / block metadata on sm_100a:
// texture fetch (TLD, the texture data pipe) vs ld.global.nc (the LSU data
// pipe) vs shared memory, as a function of how many distinct addresses one
// warp instruction touches (32, 4 or 1).  L1-resident data, 8 independent
// loads per iteration so the probe measures throughput, not latency.
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/load_probe.cu -o tools/load_probe
#include <cstdio>
#include <cuda_runtime.h>

constexpr int kN4 = 1024;  // float4 elements (16 KB, L1-resident)
constexpr int kIters = 2048;

__device__ __forceinline__ int addr_of(int mode, int lane, int i) {
    // distinct 32-byte segments (2 float4 each) per warp instruction
    const int seg = mode == 32 ? lane : mode == 4 ? (lane >> 3) : 0;
    return ((seg * 37 + i * 11) & (kN4 / 2 - 1)) * 2;
}

template <int MODE>
__global__ void k_tex(cudaTextureObject_t t, float *out) {
    const int lane = threadIdx.x & 31;
    float4 acc = make_float4(0, 0, 0, 0);
    for (int i = 0; i < kIters; i += 8) {
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const float4 v = tex1Dfetch<float4>(t, addr_of(MODE, lane, i + u) + (u & 1));
            acc.x += v.x, acc.y += v.y, acc.z += v.z, acc.w += v.w;
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc.x + acc.y + acc.z + acc.w;
}

template <int MODE>
__global__ void k_ldg256(const float *x, float *out) {
    const int lane = threadIdx.x & 31;
    float acc = 0.f;
    for (int i = 0; i < kIters; i += 8) {
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const float *p = x + 4 * addr_of(MODE, lane, i + u);
            float v[8];
            asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                         : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]),
                           "=f"(v[7])
                         : "l"(p));
            acc += ((v[0] + v[1]) + (v[2] + v[3])) + ((v[4] + v[5]) + (v[6] + v[7]));
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <int MODE>
__global__ void k_ldg32(const float *x, float *out) {
    const int lane = threadIdx.x & 31;
    float acc = 0.f;
    for (int i = 0; i < kIters; i += 8) {
#pragma unroll
        for (int u = 0; u < 8; ++u) acc += __ldg(x + 4 * addr_of(MODE, lane, i + u) + (lane & 7));
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc;
}

template <int MODE>
__global__ void k_lds128(const float *x, float *out) {
    __shared__ float4 s[kN4];
    for (int i = threadIdx.x; i < kN4; i += blockDim.x) s[i] = reinterpret_cast<const float4 *>(x)[i];
    __syncthreads();
    const int lane = threadIdx.x & 31;
    float4 acc = make_float4(0, 0, 0, 0);
    for (int i = 0; i < kIters; i += 8) {
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const float4 v = s[addr_of(MODE, lane, i + u) + (u & 1)];
            acc.x += v.x, acc.y += v.y, acc.z += v.z, acc.w += v.w;
        }
    }
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc.x + acc.y + acc.z + acc.w;
}

template <class F>
void run(const char *name, F launch, int blocks, int threads) {
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    launch();
    cudaEventRecord(a);
    for (int r = 0; r < 5; ++r) launch();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    int dev = 0, clk = 0, sms = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const double warp_instr = 5.0 * blocks * (threads / 32) * (double)kIters;
    const double sm_cycles = ms * 1e-3 * clk * 1e3;  // per SM
    printf("%-12s %8.3f ms  %6.3f SM-cycles per warp-load instruction\n", name, ms / 5,
           sm_cycles / (warp_instr / sms));
}

int main() {
    float *x, *out;
    cudaMalloc(&x, kN4 * 16);
    cudaMemset(x, 0, kN4 * 16);
    const int blocks = 148 * 8, threads = 256;
    cudaMalloc(&out, (size_t)blocks * threads * 4);
    cudaResourceDesc rd{};
    rd.resType = cudaResourceTypeLinear;
    rd.res.linear.devPtr = x;
    rd.res.linear.desc = cudaCreateChannelDesc<float4>();
    rd.res.linear.sizeInBytes = kN4 * 16;
    cudaTextureDesc td{};
    td.readMode = cudaReadModeElementType;
    cudaTextureObject_t t;
    cudaCreateTextureObject(&t, &rd, &td, nullptr);
    run("tex128_d32", [&] { k_tex<32><<<blocks, threads>>>(t, out); }, blocks, threads);
    run("tex128_d4", [&] { k_tex<4><<<blocks, threads>>>(t, out); }, blocks, threads);
    run("tex128_d1", [&] { k_tex<1><<<blocks, threads>>>(t, out); }, blocks, threads);
    run("ldg256_d32", [&] { k_ldg256<32><<<blocks, threads>>>(x, out); }, blocks, threads);
    run("ldg256_d4", [&] { k_ldg256<4><<<blocks, threads>>>(x, out); }, blocks, threads);
    run("ldg256_d1", [&] { k_ldg256<1><<<blocks, threads>>>(x, out); }, blocks, threads);
    run("ldg32_d32", [&] { k_ldg32<32><<<blocks, threads>>>(x, out); }, blocks, threads);
    run("ldg32_d4", [&] { k_ldg32<4><<<blocks, threads>>>(x, out); }, blocks, threads);
    run("ldg32_d1", [&] { k_ldg32<1><<<blocks, threads>>>(x, out); }, blocks, threads);
    run("lds128_d32", [&] { k_lds128<32><<<blocks, threads>>>(x, out); }, blocks, threads);
    run("lds128_d4", [&] { k_lds128<4><<<blocks, threads>>>(x, out); }, blocks, threads);
    run("lds128_d1", [&] { k_lds128<1><<<blocks, threads>>>(x, out); }, blocks, threads);
    cudaError_t e = cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(e));
}
