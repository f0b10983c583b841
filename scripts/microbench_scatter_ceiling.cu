// microbench_scatter_ceiling.cu -- what a 256-way radix scatter can reach on this B200:
//   copy      : read 8 B/elem sequentially, write 8 B/elem sequentially (roofline reference)
//   runs<L>   : read sequentially, write runs of L elements to 256 interleaved bucket streams
//               (each CTA owns a contiguous slice of every bucket; run alignment as produced by
//               a tile-at-a-time scatter: 8 B granularity, no line alignment)
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a scripts/microbench_scatter_ceiling.cu -o /tmp/sc && /tmp/sc
#include <cstdint>
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_copy(const uint2* __restrict__ in, uint2* __restrict__ out, uint64_t n) {
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
        out[i] = in[i];
}

// Element i of tile t (tile = 4096 elements = 256 buckets x 16) goes to bucket b = (i / L) % 256;
// bucket b of the whole array starts at b * (n / 256); within the bucket, tile t's run starts at
// t * 16 * (L / 16)... simplified: run k of bucket b written by "tile" k, length L, at offset
// b * bucket_len + k * L + skew (skew makes runs 8-byte but not line aligned).
template <int L>
__global__ void k_runs(const uint2* __restrict__ in, uint2* __restrict__ out, uint64_t n, uint32_t skew) {
    const uint64_t bucket_len = n / 256;
    for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
        const uint64_t run = i / L;             // global run id
        const uint32_t b = (uint32_t)(run % 256);
        const uint64_t k = run / 256;           // run index inside the bucket
        uint64_t dst = b * bucket_len + k * L + (i % L) + skew;
        if (dst >= n) dst -= n;
        out[dst] = in[i];
    }
}

int main() {
    const uint64_t n = 1ull << 28;  // 2 GiB per buffer
    uint2 *in, *out;
    cudaMalloc(&in, n * 8 + 4096);
    cudaMalloc(&out, n * 8 + 4096);
    cudaMemset(in, 1, n * 8);
    int sms;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    auto run = [&](const char* name, auto launch) {
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        launch();
        cudaEventRecord(a);
        for (int r = 0; r < 5; ++r) launch();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        ms /= 5;
        printf("%-22s %8.3f ms  %8.1f GB/s (16 B/elem)\n", name, ms, 16.0 * n / (ms * 1e-3) / 1e9);
    };
    const unsigned grid = sms * 8;
    run("copy", [&] { k_copy<<<grid, 512>>>(in, out, n); });
    run("runs L=8  skew=1", [&] { k_runs<8><<<grid, 512>>>(in, out, n, 1); });
    run("runs L=16 skew=1", [&] { k_runs<16><<<grid, 512>>>(in, out, n, 1); });
    run("runs L=16 skew=0", [&] { k_runs<16><<<grid, 512>>>(in, out, n, 0); });
    run("runs L=16 skew=4 (sector-aligned)", [&] { k_runs<16><<<grid, 512>>>(in, out, n, 4); });
    run("runs L=16 skew=8", [&] { k_runs<16><<<grid, 512>>>(in, out, n, 8); });
    run("runs L=32 skew=4 (sector-aligned)", [&] { k_runs<32><<<grid, 512>>>(in, out, n, 4); });
    run("runs L=32 skew=1", [&] { k_runs<32><<<grid, 512>>>(in, out, n, 1); });
    run("runs L=32 skew=0", [&] { k_runs<32><<<grid, 512>>>(in, out, n, 0); });
    run("runs L=64 skew=1", [&] { k_runs<64><<<grid, 512>>>(in, out, n, 1); });
    run("runs L=128 skew=1", [&] { k_runs<128><<<grid, 512>>>(in, out, n, 1); });
    printf("err=%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
