"""Memory skeleton of the warp-bin sweep: the same loads as k_warp2 (row
metadata, indices, weights, neighbour labels) with the fold replaced by an
XOR, to separate memory-system time from fold instructions."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch, synth
from torch.utils.cpp_extension import load_inline

src = r"""
#include <torch/extension.h>
#include <cuda_runtime.h>
template <int MODE>
__global__ void __launch_bounds__(256, 6) skel(const long* __restrict__ off, const int* __restrict__ idx, const float* __restrict__ wt,
    const int* __restrict__ lab, const int* __restrict__ list, long n, int* out) {
  const int lane = threadIdx.x & 31;
  long nw = (long)gridDim.x * 8;
  int acc = 0;
  for (long c = (long)blockIdx.x * 8 + (threadIdx.x >> 5); c < (n + 31) / 32; c += nw) {
    long t = c * 32 + lane;
    long o = 0; unsigned d = 0;
    if (t < n) { int r = list[t]; o = off[r]; d = (unsigned)(off[r + 1] - o); }
    unsigned act = __ballot_sync(~0u, d > 0);
    while (act) {
      int k = __ffs(act) - 1; act &= act - 1;
      long ok = __shfl_sync(~0u, o, k); unsigned dk = __shfl_sync(~0u, d, k);
      for (unsigned b = 0; b < dk; b += 64) {
        int j0 = b + lane < dk ? __ldcs(idx + ok + b + lane) : -1;
        int j1 = b + 32 + lane < dk ? __ldcs(idx + ok + b + 32 + lane) : -1;
        float w0 = b + lane < dk ? __ldcs(wt + ok + b + lane) : 0.f;
        float w1 = b + 32 + lane < dk ? __ldcs(wt + ok + b + 32 + lane) : 0.f;
        if (MODE == 0) { acc ^= j0 ^ j1 ^ __float_as_int(w0) ^ __float_as_int(w1); }
        else {
          int k0 = j0 >= 0 ? lab[j0] : 0, k1 = j1 >= 0 ? lab[j1] : 0;
          if (MODE == 1) acc ^= k0 ^ k1 ^ __float_as_int(w0) ^ __float_as_int(w1);
          else { unsigned g = __match_any_sync(~0u, k0); unsigned g2 = __match_any_sync(~0u, k1); acc ^= g ^ g2 ^ __float_as_int(w0); }
        }
      }
    }
  }
  if (acc == 0x12345) out[0] = acc;
}
void run(torch::Tensor off, torch::Tensor idx, torch::Tensor wt, torch::Tensor lab, torch::Tensor list, torch::Tensor out, int mode, int grid) {
  long n = list.numel();
  auto s = at::cuda::getCurrentCUDAStream();
  if (mode == 0) skel<0><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>());
  else if (mode == 1) skel<1><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>());
  else skel<2><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>());
}
"""
m = load_inline("skel", cpp_sources="void run(torch::Tensor off, torch::Tensor idx, torch::Tensor wt, torch::Tensor lab, torch::Tensor list, torch::Tensor out, int mode, int grid);",
                cuda_sources="#include <ATen/cuda/CUDAContext.h>\n" + src, functions=["run"],
                extra_cuda_cflags=["-gencode", "arch=compute_100a,code=sm_100a", "-O3"], verbose=False)
g = synth.make("web_40m_2200m", device="cuda")
deg = g.offsets[1:] - g.offsets[:-1]
rows = torch.nonzero((deg >= 16) & (deg < 256)).flatten().to(torch.int32)
w = torch.ones(g.M, device="cuda", dtype=torch.float32)
import paper_conf_ipps_sahunk25_b200 as nl
gg = nl.Graph(g.offsets, g.indices, w)
gg.run()
labels = gg.labels().clone()
out = torch.zeros(1, dtype=torch.int32, device="cuda")
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for mode, name in ((0, "stream idx+w"), (1, "+ label gather"), (2, "+ gather + 2 match_any")):
    for grid in (148 * 6,):
        ts = []
        for r in range(4):
            torch.cuda.synchronize(); e0.record()
            m.run(g.offsets, g.indices, w, labels, rows, out, mode, grid)
            e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
        print(f"{name:28s} grid {grid}: {min(ts):.3f} ms", flush=True)
