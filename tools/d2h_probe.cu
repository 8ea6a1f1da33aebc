// d2h_probe.cu -- host-link (PCIe) D2H behaviour under the pipeline's patterns (diagnostic tool).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o d2h_probe d2h_probe.cu
// Prints one JSON object: GB/s for copy-engine D2H with various chunkings / streams, and for SM
// stores straight into mapped pinned host memory (zero-copy), the alternative to the ring + copy.
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x)                                                                        \
    do {                                                                             \
        cudaError_t e = (x);                                                         \
        if (e != cudaSuccess) {                                                      \
            fprintf(stderr, "%s:%d %s: %s\n", __FILE__, __LINE__, #x, cudaGetErrorString(e)); \
            exit(1);                                                                 \
        }                                                                            \
    } while (0)

__global__ void k_store(const int4 *__restrict__ src, int4 *__restrict__ dst, size_t n16) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n16; i += (size_t)gridDim.x * blockDim.x)
        dst[i] = src[i];
}

int main() {
    const size_t N = 3058081248ull;  // 12 B x nnz(C2)
    char *d, *h, *h2;
    CK(cudaMalloc(&d, N));
    CK(cudaMemset(d, 1, N));
    CK(cudaHostAlloc(&h, N, cudaHostAllocMapped));
    CK(cudaHostAlloc(&h2, N, 0));
    cudaStream_t s1, s2;
    CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
    CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    auto run = [&](auto fn) {
        float best = 1e30f;
        for (int r = 0; r < 4; ++r) {
            CK(cudaDeviceSynchronize());
            CK(cudaEventRecord(a, s1));
            fn();
            CK(cudaEventRecord(b, s1));
            CK(cudaEventSynchronize(b));
            float ms;
            CK(cudaEventElapsedTime(&ms, a, b));
            if (r > 0 && ms < best) best = ms;
        }
        return N / (best * 1e6);
    };
    printf("{\n");
    printf(" \"single_copy_GBps\": %.2f,\n", run([&] { CK(cudaMemcpyAsync(h2, d, N, cudaMemcpyDeviceToHost, s1)); }));
    for (int nc : {2, 8, 22, 44, 128}) {
        printf(" \"chunks_%d_one_stream_GBps\": %.2f,\n", nc, run([&] {
                   size_t step = (N / nc + 255) & ~size_t(255);
                   for (size_t o = 0; o < N; o += step)
                       CK(cudaMemcpyAsync(h2 + o, d + o, (o + step < N ? step : N - o), cudaMemcpyDeviceToHost, s1));
               }));
    }
    printf(" \"chunks_44_two_streams_GBps\": %.2f,\n", run([&] {
               size_t step = (N / 44 + 255) & ~size_t(255);
               int k = 0;
               for (size_t o = 0; o < N; o += step, ++k)
                   CK(cudaMemcpyAsync(h2 + o, d + o, (o + step < N ? step : N - o), cudaMemcpyDeviceToHost, (k & 1) ? s2 : s1));
               CK(cudaEventRecord(b, s2));
               CK(cudaStreamWaitEvent(s1, b, 0));
           }));
    printf(" \"single_copy_mapped_dst_GBps\": %.2f,\n", run([&] { CK(cudaMemcpyAsync(h, d, N, cudaMemcpyDeviceToHost, s1)); }));
    int4 *hd;
    CK(cudaHostGetDevicePointer((void **)&hd, h, 0));
    for (int blocks : {148, 296, 592, 1184}) {
        printf(" \"zero_copy_sm_stores_%d_blocks_GBps\": %.2f,\n", blocks, run([&] {
                   k_store<<<blocks, 512, 0, s1>>>((const int4 *)d, hd, N / 16);
               }));
    }
    printf(" \"done\": 1\n}\n");
    return 0;
}
