// spin.cu — TEST HELPER ONLY (not product code): a kernel that occupies SMs for a while, so
// tests can launch libbar's solves while other work holds most of the device.
#include <cuda_runtime.h>

__global__ void k_spin(unsigned long long ns) {
    extern __shared__ unsigned char pad[];
    if (threadIdx.x == 0) {
        unsigned long long t0, t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        do {
            __nanosleep(1000);
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        } while (t - t0 < ns);
        pad[0] = 1;
    }
    __syncthreads();
}

// blocks x threads with smem_bytes of dynamic shared memory each, spinning for ns nanoseconds
extern "C" int spin_launch(int blocks, int threads, int smem_bytes, unsigned long long ns, void *stream) {
    if (cudaFuncSetAttribute(k_spin, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes) != cudaSuccess)
        return (int)cudaGetLastError();
    k_spin<<<blocks, threads, smem_bytes, (cudaStream_t)stream>>>(ns);
    return (int)cudaGetLastError();
}

extern "C" int spin_sm_count(int device) {
    int v = 0;
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, device);
    return v;
}
