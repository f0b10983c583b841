// microbench_warp_ops.cu -- throughput of the warp primitives the partition kernels can rank /
// count with on sm_100a: MATCH.ANY, ballot-built match, shared-memory atomics (spread / colliding,
// with and without return).  Reports SM-cycles per warp-instruction-equivalent (full chip).
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a scripts/microbench_warp_ops.cu -o /tmp/mb && /tmp/mb
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t lcg(uint32_t x) { return x * 1664525u + 1013904223u; }

template <int MODE>
__global__ void __launch_bounds__(1024) k(uint32_t iters, uint32_t* out, uint32_t bins_mask) {
    extern __shared__ uint32_t sh[];
    for (uint32_t i = threadIdx.x; i <= bins_mask; i += blockDim.x) sh[i] = 0;
    __syncthreads();
    uint32_t x = lcg(threadIdx.x * 7919u + blockIdx.x * 104729u);
    uint32_t acc = 0;
    const uint32_t lane = threadIdx.x & 31;
    uint32_t lt;
    asm("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
    for (uint32_t it = 0; it < iters; ++it) {
        x = lcg(x);
        uint32_t v = (x >> 8) & bins_mask;
        if (MODE == 0) {  // match.any
            acc += __match_any_sync(0xffffffffu, v);
        } else if (MODE == 1) {  // ballot match on 16 bits
            uint32_t m = 0xffffffffu;
#pragma unroll
            for (int b = 0; b < 16; ++b) {
                uint32_t bb = __ballot_sync(0xffffffffu, (v >> b) & 1);
                m &= ((v >> b) & 1) ? bb : ~bb;
            }
            acc += m;
        } else if (MODE == 2) {  // ballot match on 8 bits
            uint32_t m = 0xffffffffu;
#pragma unroll
            for (int b = 0; b < 8; ++b) {
                uint32_t bb = __ballot_sync(0xffffffffu, (v >> b) & 1);
                m &= ((v >> b) & 1) ? bb : ~bb;
            }
            acc += m;
        } else if (MODE == 3) {  // ATOMS.ADD no return, spread
            atomicAdd(&sh[v], 1u);
        } else if (MODE == 4) {  // ATOMS.ADD with return, spread
            acc += atomicAdd(&sh[v], 1u);
        } else if (MODE == 5) {  // ATOMS all lanes same address
            atomicAdd(&sh[(x >> 20) & 7 & bins_mask], 1u);
        } else if (MODE == 6) {  // match + leader atomic (hist style)
            uint32_t p = __match_any_sync(0xffffffffu, v);
            if ((p & lt) == 0) atomicAdd(&sh[v], __popc(p));
        } else if (MODE == 7) {  // plain ALU baseline (lcg only)
            acc += v;
        } else if (MODE == 8) {  // ATOMS.ADD no return, warp-uniform address
            atomicAdd(&sh[__shfl_sync(0xffffffffu, v, 0)], 1u);
        } else if (MODE == 9) {  // packed u16 counters (2 bins per word), with return (wrap check)
            const uint32_t vv = (x >> 8) & (2 * bins_mask + 1);
            const uint32_t sh16 = (vv & 1) << 4;
            const uint32_t old = atomicAdd(&sh[vv >> 1], 1u << sh16);
            acc += ((old >> sh16) & 0xffffu) == 0xffffu;
        } else if (MODE == 10) {  // packed u16, colliding (8 bins)
            const uint32_t vv = (x >> 20) & 7;
            const uint32_t sh16 = (vv & 1) << 4;
            const uint32_t old = atomicAdd(&sh[vv >> 1], 1u << sh16);
            acc += ((old >> sh16) & 0xffffu) == 0xffffu;
        } else if (MODE == 11) {  // packed u16, all lanes one bin
            const uint32_t old = atomicAdd(&sh[3], 1u << 16);
            acc += (old >> 16) == 0xffffu;
        } else if (MODE == 12) {  // u32, all lanes one bin, +1 no return
            atomicAdd(&sh[3], 1u);
        }
    }
    __syncthreads();
    if (acc == 0x12345678u) out[0] = acc + sh[lane];
    if (threadIdx.x == 0) out[1 + blockIdx.x] = sh[0];
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    int clk = 0;
    cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
    uint32_t* out;
    cudaMalloc(&out, 4096 * 4);
    const char* names[] = {"match.any(16b)", "ballot-match 16b", "ballot-match 8b", "atoms.add spread",
                           "atoms.add ret spread", "atoms.add collide(8 addr)", "match+leader atom", "alu baseline",
                           "atoms uniform addr", "packed16 ret spread", "packed16 ret collide8", "packed16 ret one bin", "atoms +1 one bin"};
    void (*fns[])(uint32_t, uint32_t*, uint32_t) = {k<0>, k<1>, k<2>, k<3>, k<4>, k<5>, k<6>, k<7>, k<8>, k<9>, k<10>, k<11>, k<12>};
    const uint32_t iters = 4096;
    for (int m = 3; m < 13; ++m) {
        for (uint32_t mask : {0xffffu >> 1, 0xffu}) {
            size_t smem = size_t(mask + 1) * 4;
            cudaFuncSetAttribute(fns[m], cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
            cudaEvent_t a, b;
            cudaEventCreate(&a);
            cudaEventCreate(&b);
            fns[m]<<<sms, 1024, smem>>>(iters, out, mask);
            cudaEventRecord(a);
            fns[m]<<<sms, 1024, smem>>>(iters, out, mask);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            float ms;
            cudaEventElapsedTime(&ms, a, b);
            double warp_ops_per_sm = 32.0 * iters;  // 32 warps per CTA, 1 CTA per SM
            double cycles = ms * 1e-3 * clk * 1e3;
            printf("%-28s bins=%6u  %8.3f ms  %6.2f SM-cycles per warp-op  (%.1f G lane-ops/s chip)\n", names[m],
                   mask + 1, ms, cycles / warp_ops_per_sm, 32.0 * warp_ops_per_sm * sms / (ms * 1e-3) / 1e9);
        }
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("err=%s clk=%d kHz sms=%d\n", cudaGetErrorString(e), clk, sms);
    return 0;
}
