// Probe: does SHFL consume L1/shared data-pipe wavefronts? (ncu metrics)
#include <cstdio>
__global__ void k_shfl(float *out, int iters) {
    float v = threadIdx.x;
    for (int i = 0; i < iters; ++i) v += __shfl_sync(0xffffffffu, v, (threadIdx.x * 7 + i) & 31);
    out[blockIdx.x * blockDim.x + threadIdx.x] = v;
}
__global__ void k_lds(float *out, int iters) {
    __shared__ float s[1024];
    s[threadIdx.x] = threadIdx.x;
    __syncthreads();
    float v = 0;
    for (int i = 0; i < iters; ++i) v += s[(threadIdx.x * 7 + i) & 1023];
    out[blockIdx.x * blockDim.x + threadIdx.x] = v;
}
int main() {
    float *o;
    cudaMalloc(&o, 148 * 8 * 1024 * 4);
    k_shfl<<<148 * 8, 1024>>>(o, 4096);
    k_lds<<<148 * 8, 1024>>>(o, 4096);
    cudaDeviceSynchronize();
    printf("ok\n");
}
