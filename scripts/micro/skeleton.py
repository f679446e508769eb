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
__global__ void __launch_bounds__(256, MODE >= 3 ? 4 : 8) skel(const long* __restrict__ off, const int* __restrict__ idx, const float* __restrict__ wt,
    const int* __restrict__ lab, const int* __restrict__ list, long n, int* out, int contig) {
  const int lane = threadIdx.x & 31;
  long nw = (long)gridDim.x * 8;
  int acc = 0;
  const long nc = (n + 31) / 32, gw = (long)blockIdx.x * 8 + (threadIdx.x >> 5);
  const long c0 = contig ? gw * nc / nw : gw, c1 = contig ? (gw + 1) * nc / nw : nc, cs = contig ? 1 : nw;
  for (long c = c0; c < c1; c += cs) {
    long t = c * 32 + lane;
    long o = 0; unsigned d = 0;
    if (t < n) { int r = list[t]; o = off[r]; d = (unsigned)(off[r + 1] - o); }
    unsigned act = __ballot_sync(~0u, d > 0);
    if (MODE == 7 || MODE == 8) {
      // chunk-pipelined: the sequence of 64-entry chunks of the 32 rows
      // (MODE 8: entries past 64 skipped -- upper bound), loads of chunk
      // c+2, gathers of chunk c+1, consume chunk c
      auto nch = [&](int k) -> int { unsigned dk = __shfl_sync(~0u, d, k & 31); return k >= 32 ? 1 : (MODE == 8 ? 1 : (int)max(1u, (dk + 63) / 64)); };
      auto ldc = [&](int k, int c, int* jj) {
        long ok = __shfl_sync(~0u, o, k & 31); unsigned dk = __shfl_sync(~0u, d, k & 31);
        if (k >= 32) dk = 0;
        unsigned b = 64u * c;
        jj[0] = b + lane < dk ? __ldcs(idx + ok + b + lane) : -1;
        jj[1] = b + 32 + lane < dk ? __ldcs(idx + ok + b + 32 + lane) : -1;
      };
      auto gat = [&](const int* jj, int* kk) { kk[0] = jj[0] >= 0 ? lab[jj[0]] : 0; kk[1] = jj[1] >= 0 ? lab[jj[1]] : 0; };
      // stage positions (row, chunk)
      int k0 = 0, c0 = 0;
      int k1 = k0, c1 = c0; if (++c1 >= nch(k1)) { ++k1; c1 = 0; }
      int k2 = k1, c2 = c1; if (++c2 >= nch(k2)) { ++k2; c2 = 0; }
      int J0[2], J1[2], J2[2], K0[2], K1[2];
      ldc(k0, c0, J0); ldc(k1, c1, J1); gat(J0, K0);
      while (k0 < 32) {
        ldc(k2, c2, J2);
        gat(J1, K1);
        acc ^= K0[0] ^ K0[1];
        k0 = k1; c0 = c1; k1 = k2; c1 = c2;
        if (++c2 >= nch(k2)) { ++k2; c2 = 0; }
        J0[0] = J1[0]; J0[1] = J1[1]; J1[0] = J2[0]; J1[1] = J2[1]; K0[0] = K1[0]; K0[1] = K1[1];
      }
      continue;
    }
    if (MODE == 9 && c + cs < c1) {
      // bulk L2 prefetch of the NEXT chunk's CSR index span (one instruction)
      if (lane == 0) {
        long tn = (c + cs) * 32;
        int r0 = list[tn], r1 = list[min(tn + 31, n - 1)];
        long b0 = off[r0] & ~3L, b1 = (off[r1 + 1] + 3) & ~3L;
        unsigned bytes = (unsigned)((b1 - b0) * 4);
        if (bytes >= 16) asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(idx + b0), "r"(bytes) : "memory");
      }
    }
    if (MODE >= 3) {
      // software-pipelined: at vertex k, index loads of k+D+1, gathers of k+D, consume k
      constexpr int D = MODE >= 3 && MODE <= 6 ? MODE - 2 : 1;
      int J[D + 2][2]; int K[D + 1][2];
      auto ldidx = [&](int k, int* jj) {
        long ok = __shfl_sync(~0u, o, k & 31); unsigned dk = __shfl_sync(~0u, d, k & 31);
        if (k >= 32) dk = 0;
        jj[0] = lane < dk ? __ldcs(idx + ok + lane) : -1;
        jj[1] = lane + 32 < dk ? __ldcs(idx + ok + 32 + lane) : -1;
      };
      auto gat = [&](const int* jj, int* kk) { kk[0] = jj[0] >= 0 ? lab[jj[0]] : 0; kk[1] = jj[1] >= 0 ? lab[jj[1]] : 0; };
#pragma unroll
      for (int s = 0; s <= D; ++s) ldidx(s, J[s]);
#pragma unroll
      for (int s = 0; s < D; ++s) gat(J[s], K[s]);
      for (int k = 0; k < 32; ++k) {
        ldidx(k + D + 1, J[D + 1]);
        gat(J[D], K[D]);
        acc ^= K[0][0] ^ K[0][1];
        // rest of row k (entries 64..), unpipelined
        long ok = __shfl_sync(~0u, o, k); unsigned dk = __shfl_sync(~0u, d, k);
        for (unsigned b = 64; b < dk; b += 64) {
          int j0 = b + lane < dk ? __ldcs(idx + ok + b + lane) : -1;
          int j1 = b + 32 + lane < dk ? __ldcs(idx + ok + b + 32 + lane) : -1;
          acc ^= (j0 >= 0 ? lab[j0] : 0) ^ (j1 >= 0 ? lab[j1] : 0);
        }
#pragma unroll
        for (int s = 0; s < D; ++s) { K[s][0] = K[s + 1][0]; K[s][1] = K[s + 1][1]; }
#pragma unroll
        for (int s = 0; s <= D; ++s) { J[s][0] = J[s + 1][0]; J[s][1] = J[s + 1][1]; }
      }
      continue;
    }
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
void run(torch::Tensor off, torch::Tensor idx, torch::Tensor wt, torch::Tensor lab, torch::Tensor list, torch::Tensor out, int mode, int grid, int contig) {
  long n = list.numel();
  auto s = at::cuda::getCurrentCUDAStream();
  if (mode == 0) skel<0><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
  else if (mode == 1) skel<1><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
  else if (mode == 2) skel<2><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
  else if (mode == 3) skel<3><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
  else if (mode == 4) skel<4><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
  else if (mode == 7) skel<7><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
  else if (mode == 9) skel<9><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
  else if (mode == 8) skel<8><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
  else skel<6><<<grid, 256, 0, s>>>(off.data_ptr<long>(), idx.data_ptr<int>(), wt.data_ptr<float>(), lab.data_ptr<int>(), list.data_ptr<int>(), n, out.data_ptr<int>(), contig);
}
"""
m = load_inline("skel", cpp_sources="void run(torch::Tensor off, torch::Tensor idx, torch::Tensor wt, torch::Tensor lab, torch::Tensor list, torch::Tensor out, int mode, int grid, int contig);",
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
MODES = [int(x) for x in os.environ.get("SKEL_MODES", "0,1,2").split(",")]
NAMES = {0: "stream idx+w", 1: "+ label gather", 2: "+ gather + 2 match_any", 3: "pipelined idx, gather lead 1", 4: "pipelined, gather lead 2", 6: "pipelined, gather lead 4", 7: "chunk-pipelined lead 1", 8: "first 64 entries only (bound)", 9: "pipelined + next-chunk L2 prefetch"}
for mode, name in [(m, NAMES[m]) for m in MODES]:
    for grid, contig in [(g, c) for g, c in ((148 * 4, 0), (148 * 6, 0), (148 * 8, 0), (148 * 4, 1), (148 * 8, 1)) if mode < 3 or g == 148 * 4]:
        ts = []
        for r in range(4):
            torch.cuda.synchronize(); e0.record()
            m.run(g.offsets, g.indices, w, labels, rows, out, mode, grid, contig)
            e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
        print(f"{name:28s} grid {grid} contig {contig}: {min(ts):.3f} ms", flush=True)

# sweep-0 schedule in phases: the contiguous-run schedule applied to P
# consecutive slices of the bin one after another (smaller label window per
# phase, runs 1/P as long)
if os.environ.get("SKEL_PHASES"):
    for mode in (3,):
        for P in [int(x) for x in os.environ["SKEL_PHASES"].split(",")]:
            ts = []
            n = rows.numel()
            for r in range(3):
                torch.cuda.synchronize(); e0.record()
                for p in range(P):
                    sl = rows[p * n // P:(p + 1) * n // P]
                    m.run(g.offsets, g.indices, w, labels, sl, out, mode, 148 * 4, 1)
                e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
            print(f"{NAMES[mode]:28s} contiguous runs in {P} phases: {min(ts):.3f} ms", flush=True)
