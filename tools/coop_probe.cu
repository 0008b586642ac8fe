// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o coop_probe tools/coop_probe.cu (run on a B200).
// probe: can two cooperative kernels on two streams of one process run concurrently?
#include <cooperative_groups.h>
#include <cstdio>
namespace cg = cooperative_groups;
__global__ void k(int me, int* flags, unsigned long long cap, int* result) {
    cg::grid_group g = cg::this_grid();
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        atomicExch(flags + me, 1);
        unsigned long long s = 0;
        while (atomicAdd(flags + (1 - me), 0) == 0 && ++s < cap) __nanosleep(100);
        result[me] = (s < cap) ? 1 : -1;
    }
    g.sync();
}
int main() {
    int *flags, *res;
    cudaMalloc(&flags, 8); cudaMemset(flags, 0, 8);
    cudaMalloc(&res, 8); cudaMemset(res, 0, 8);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaStream_t s0, s1; cudaStreamCreateWithFlags(&s0, cudaStreamNonBlocking); cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking);
    unsigned long long cap = 20000000ull;   // ~2 s of 100 ns sleeps
    int me0 = 0, me1 = 1;
    void* a0[] = {&me0, &flags, &cap, &res};
    void* a1[] = {&me1, &flags, &cap, &res};
    cudaError_t e0 = cudaLaunchCooperativeKernel((void*)k, dim3(sms), dim3(256), a0, 0, s0);
    cudaError_t e1 = cudaLaunchCooperativeKernel((void*)k, dim3(sms), dim3(256), a1, 0, s1);
    cudaError_t e2 = cudaDeviceSynchronize();
    int h[2]; cudaMemcpy(h, res, 8, cudaMemcpyDeviceToHost);
    printf("launch %d %d sync %d results %d %d (1 = saw the other kernel, -1 = cap hit)\n", e0, e1, e2, h[0], h[1]);
    return 0;
}
