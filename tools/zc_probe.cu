// Zero-copy write probe (diagnostic): throughput of SM stores into mapped pinned host memory over
// the host link, for (a) one contiguous stream, (b) row pieces of L bytes at gapped offsets (the
// pattern of C[i][j] row pieces landing at their final host CSR positions when B is cut into
// column panels), vs the copy engine.  Prints one JSON line.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("err %s line %d\n", cudaGetErrorString(e), __LINE__); return 1; } } while (0)

__global__ void k_contig(const double2 *__restrict__ src, double2 *dst, size_t n) {
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) dst[i] = src[i];
}
// one warp per piece; piece p: src [soff[p], soff[p]+len[p]) doubles -> dst at doff[p]
__global__ void k_pieces(const double *__restrict__ src, double *dst, const int64_t *soff, const int64_t *doff,
                         const int *len, int np) {
    const int lane = threadIdx.x & 31;
    for (int p = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; p < np; p += (gridDim.x * blockDim.x) >> 5) {
        const int64_t s = soff[p], d = doff[p];
        const int L = len[p];
        for (int k = lane; k < L; k += 32) dst[d + k] = src[s + k];
    }
}

int main() {
    const size_t bytes = size_t(2) << 30;
    double *dsrc, *hdst, *hdev;
    CK(cudaMalloc(&dsrc, bytes));
    CK(cudaMemset(dsrc, 1, bytes));
    CK(cudaHostAlloc(&hdst, bytes * 3, cudaHostAllocMapped));
    CK(cudaHostGetDevicePointer((void **)&hdev, hdst, 0));
    for (size_t i = 0; i < bytes * 3 / 8; i += 512) hdst[i] = 0;  // touch
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    auto tm = [&](auto f) { float best = 1e9; for (int r = 0; r < 3; ++r) { cudaEventRecord(e0); f(); cudaEventRecord(e1); cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1); if (ms < best) best = ms; } return best; };
    printf("{");
    float ms = tm([&] { cudaMemcpyAsync(hdst, dsrc, bytes, cudaMemcpyDeviceToHost); });
    printf("\"copy_engine_GBps\": %.2f", bytes / ms / 1e6);
    for (int bl : {1, 2, 4, 8}) {
        ms = tm([&] { k_contig<<<sms * bl, 256>>>((const double2 *)dsrc, (double2 *)hdev, bytes / 16); });
        printf(", \"zc_contig_%dx_GBps\": %.2f", bl, bytes / ms / 1e6);
    }
    // pieces: lengths in doubles ~ U[lo, hi], gapped (panels = g): dst offset advances by len * g
    for (int lo : {8, 40, 120}) for (int g : {1, 2, 4}) {
        std::vector<int64_t> so, dof; std::vector<int> ln;
        uint64_t x = 12345; int64_t s = 0, d = 0;
        while (true) {
            x = x * 6364136223846793005ull + 1442695040888963407ull;
            int L = lo + int((x >> 33) % (unsigned)(lo + 1));
            if ((s + L) * 8 > (int64_t)bytes) break;
            so.push_back(s); dof.push_back(d); ln.push_back(L);
            s += L; d += int64_t(L) * g;
        }
        int np = (int)so.size();
        int64_t *dso, *ddo; int *dl;
        CK(cudaMalloc(&dso, np * 8)); CK(cudaMalloc(&ddo, np * 8)); CK(cudaMalloc(&dl, np * 4));
        CK(cudaMemcpy(dso, so.data(), np * 8, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(ddo, dof.data(), np * 8, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(dl, ln.data(), np * 4, cudaMemcpyHostToDevice));
        for (int bl : {4, 16}) {
            ms = tm([&] { k_pieces<<<sms * bl, 256>>>(dsrc, hdev, dso, ddo, dl, np); });
            printf(", \"zc_pieces_len%d-%d_gap%d_%dx_GBps\": %.2f", lo * 8, lo * 16, g, bl, s * 8.0 / ms / 1e6);
        }
        cudaFree(dso); cudaFree(ddo); cudaFree(dl);
    }
    CK(cudaGetLastError());
    printf("}\n");
    return 0;
}
