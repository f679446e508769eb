// Microbenchmark: cost of __match_any_sync vs number of distinct keys in the
// warp, and of a shared-memory slot claim by atom.shared.cas vs a plain
// store + verify.  32 warps per SM (4 CTAs x 8 warps), all SMs; reports
// clock cycles per warp-instruction-iteration.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mc scripts/micro/match_cost.cu && /tmp/mc
#include <cstdio>
#include <cstdint>

__global__ void k_match(int distinct, int iters, unsigned long long *out, int *sink) {
    const int lane = threadIdx.x & 31;
    int key = (lane % distinct) * 7919 + blockIdx.x;
    unsigned acc = 0;
    __syncthreads();
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        unsigned g = __match_any_sync(0xFFFFFFFFu, key);
        acc += g;
        key += (int)(acc & 1) * 0;   // keep dependence chain honest
        key ^= (int)(g >> 31) & 0;
    }
    long long t1 = clock64();
    if (lane == 0 && threadIdx.x == 0) atomicAdd(out, (unsigned long long)(t1 - t0));
    if (acc == 12345) sink[0] = acc;
}

// MODE 0: CAS claim of 32 distinct slots; MODE 1: STS key + syncwarp + LDS verify + STS value;
// MODE 2: LDS.64 probe only
template <int MODE>
__global__ void k_claim(int iters, unsigned long long *out, int *sink) {
    __shared__ uint32_t tab[8][1024];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int s = lane; s < 1024; s += 32) tab[wid][s] = 0xFFFFFFFFu;
    __syncthreads();
    unsigned acc = 0;
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        const uint32_t slot = ((lane * 97 + i * 31) & 511) * 2;
        const uint32_t key = lane + i * 32;
        uint32_t addr = (uint32_t)__cvta_generic_to_shared(&tab[wid][slot]);
        if (MODE == 0) {
            uint32_t old;
            asm volatile("atom.shared.cas.b32 %0, [%1], %2, %3;" : "=r"(old) : "r"(addr), "r"(0xFFFFFFFFu), "r"(key) : "memory");
            acc += old;
            asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(0xFFFFFFFFu) : "memory");
        } else if (MODE == 1) {
            asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr), "r"(key) : "memory");
            __syncwarp();
            uint32_t v;
            asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr) : "memory");
            acc += v == key;
            asm volatile("st.shared.u32 [%0], %1;" ::"r"(addr + 4), "r"(key) : "memory");
        } else {
            uint64_t v;
            asm volatile("ld.shared.u64 %0, [%1];" : "=l"(v) : "r"(addr) : "memory");
            acc += (uint32_t)v;
        }
        __syncwarp();
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) atomicAdd(out, (unsigned long long)(t1 - t0));
    if (acc == 12345) sink[0] = acc;
}

int main() {
    unsigned long long *d_out;
    int *sink;
    cudaMalloc(&d_out, 8);
    cudaMalloc(&sink, 4);
    const int blocks = 148 * 4, iters = 4096;
    for (int distinct : {1, 2, 4, 8, 16, 32}) {
        cudaMemset(d_out, 0, 8);
        k_match<<<blocks, 256>>>(distinct, iters, d_out, sink);
        unsigned long long h;
        cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
        printf("match_any distinct=%2d: %.2f cycles per warp-iteration (32 warps/SM resident, per-warp latency view)\n",
               distinct, (double)h / blocks / iters);
    }
    const char *names[3] = {"CAS claim + reset", "STS key + syncwarp + LDS verify + STS value", "LDS.64 probe"};
    for (int m = 0; m < 3; ++m) {
        cudaMemset(d_out, 0, 8);
        if (m == 0) k_claim<0><<<blocks, 256>>>(iters, d_out, sink);
        if (m == 1) k_claim<1><<<blocks, 256>>>(iters, d_out, sink);
        if (m == 2) k_claim<2><<<blocks, 256>>>(iters, d_out, sink);
        unsigned long long h;
        cudaMemcpy(&h, d_out, 8, cudaMemcpyDeviceToHost);
        printf("%s: %.2f cycles per warp-iteration\n", names[m], (double)h / blocks / iters);
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(e));
    return 0;
}
