// Microbenchmark: 4736 warps (148 SMs x 4 CTAs x 8 warps) each read R rows of
// ~53 int32 entries (212 B) from a large array.  "region": warp w's rows are
// consecutive in its own region (region = array / nw) -- the block-cyclic
// schedule's CSR stream; "interleaved": row t of warp w sits at position
// t*nw + w -- all warps read one narrow window at any time.  Same bytes.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/sl scripts/micro/stream_layout.cu && /tmp/sl
#include <cstdio>
#include <cstdint>

// GATHER: each entry also gathers lab[(vertex + d) mod nv] with a pseudo-random
// log-uniform distance d < 2^19 (host-local neighbours), vertex = the row's
// vertex id under the "schedule" (region: vertex = row; interleaved: vertex
// = the row a K=1 schedule would process at that time) -- i.e. the label
// gathers follow the processing order, the streams follow the layout.
template <bool INTERLEAVED, bool GATHER>
__global__ void __launch_bounds__(256, 4) k(const int *__restrict__ a, const int *__restrict__ lab, int64_t nv,
                                            int64_t rows_per_warp, int row_len, int *out) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = (int64_t)gridDim.x * 8, w = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
    int acc = 0;
    for (int64_t t = 0; t < rows_per_warp; ++t) {
        const int64_t row = INTERLEAVED ? t * nw + w : w * rows_per_warp + t;
        const int *p = a + row * row_len;
        int x0 = lane < row_len ? __ldcs(p + lane) : 0;
        int x1 = lane + 32 < row_len ? __ldcs(p + 32 + lane) : 0;
        if (GATHER) {
            const int64_t v = row * (nv / (rows_per_warp * nw));
            uint32_t h0 = (uint32_t)(row * 2654435761u + lane * 40503u), h1 = h0 * 747796405u + 2891336453u;
            const int64_t d0 = (int64_t)(1u << (h0 % 19)) + (h0 >> 13) % (1u << (h0 % 19));
            const int64_t d1 = (int64_t)(1u << (h1 % 19)) + (h1 >> 13) % (1u << (h1 % 19));
            if (lane < row_len) x0 ^= lab[(v + d0) % nv];
            if (lane + 32 < row_len) x1 ^= lab[(v + d1) % nv];
        }
        acc ^= x0 ^ x1;
    }
    if (acc == 0x12345678) out[0] = acc;
}

int main() {
    const int row_len = 53;
    const int blocks = 148 * 4;
    const int64_t nw = blocks * 8;
    const int64_t total = (int64_t)2 << 30;   // 2 Gi ints = 8 GiB
    const int64_t rows = total / row_len, rpw = rows / nw;
    int *a, *out;
    if (cudaMalloc(&a, total * sizeof(int)) != cudaSuccess) { printf("alloc failed\n"); return 1; }
    cudaMalloc(&out, 4);
    cudaMemset(a, 1, total * sizeof(int));
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    const int64_t nv = 40000000;
    int *lab;
    cudaMalloc(&lab, nv * sizeof(int));
    cudaMemset(lab, 2, nv * sizeof(int));
    for (int rep = 0; rep < 2; ++rep) {
        for (int mode = 0; mode < 4; ++mode) {
            cudaEventRecord(e0);
            if (mode == 0) k<false, false><<<blocks, 256>>>(a, lab, nv, rpw, row_len, out);
            if (mode == 1) k<true, false><<<blocks, 256>>>(a, lab, nv, rpw, row_len, out);
            if (mode == 2) k<false, true><<<blocks, 256>>>(a, lab, nv, rpw, row_len, out);
            if (mode == 3) k<true, true><<<blocks, 256>>>(a, lab, nv, rpw, row_len, out);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms;
            cudaEventElapsedTime(&ms, e0, e1);
            const double bytes = (double)rpw * nw * row_len * 4;
            const char *nm[4] = {"region", "interleaved", "region+gather", "interl+gather"};
            printf("%-14s %.3f ms  %.0f GB/s (stream bytes)\n", nm[mode], ms, bytes / ms / 1e6);
        }
    }
    printf("%s\n", cudaGetErrorString(cudaDeviceSynchronize()));
    return 0;
}
