// nulpa.cu -- B200 (sm_100a) implementation of the nu-LPA hot path behind the
// C ABI declared in include/nulpa.h.
//
// Paper: PAPER.md (Sahu, nu-LPA).  Algorithm 1 is the
// sweep/loop structure, Algorithm 2 the per-vertex
// hashtable, Eq. 1 the modularity.  Readings R1..R13 are
// listed in DESIGN.md.  This file shares no code with oracle/.
//
// Layout in HBM:
//   offsets  int64 [n_rows+1]   indices int32 [M]   weights float32 [M] | null
//   labels   int32 [n_global]   flags   uint8 [n_global] (1 = unprocessed)
//   bin lists int32 (row ids), one per degree bin, stable in row order
//   giant tables: int32 keys / float32 values / int32 occupied-slot lists,
//   one region of p1 = nextPow2(D)-1 slots per giant vertex.
//
// Kernels of one sweep (lpaMove): thread bin, then the warp bin on a
// high-priority stream with block + giant on a low-priority stream filling its
// tail (bin_order 3; bin_order 1 = thread -> warp -> block -> giant in order
// on the handle's stream, hubs last; bin_order 4, the default, picks 3 when
// the warp bin holds >= 2/3 of the CSR entries, else 1):
//   k_giant_snapshot / [k_giant_count] / k_giant_accumulate / k_giant_decide / k_giant_finish
//             chunked CTAs per vertex, global-memory tables
//   k_frontier + k_block   one CTA per vertex (4 or 8 warps), TMA row staging,
//                          shared-memory table (<= 2047 slots)
//   k_frontier + k_warp    compacted frontier; one warp per vertex, pipelined,
//                          epoch-tagged shared-memory table (<= 511 slots)
//   k_thread  one thread per vertex, labels in registers (degree < 16), or
//   k_tscan + k_tact       the same over a compacted frontier (asynchronous
//                          bulk bins of degree <= 8: road, k-mer)
// Past the first sweep, a vertex whose own label holds a strict majority of
// its (unit) neighbour weights skips the table fold (the majority shortcut).

#include "nulpa.h"

#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <type_traits>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

namespace {

constexpr int32_t kEmpty = -1;           // phi
constexpr int kMaxRetries = 16;          // R5
constexpr int kMaxIter = 64;             // counters kept per iteration
constexpr int kCtr = 32;                 // counters per iteration
constexpr int kCtrTScan = 24;            // counter slots 24..31: thread-bin compaction, one per wave
constexpr int kCtrRecs = 20;             // counter slot: warp-bin frontier size
constexpr int kCtrRecsW = 21;            // counter slot: block-bin frontier, warp-per-vertex part
constexpr int kCtrRecsB = 22;            // counter slot: block-bin frontier, CTA-per-vertex part
constexpr int kCtrSchedW = 17;           // counter slot: dynamic schedule of the warp-bin k_warp
constexpr int kCtrSchedB = 18;           // counter slot: dynamic schedule of the wide k_warp
// counter slots: 0 dN, 1+b processed, 5+b edges, 9+b changed, 13+b edges of changed (b = bin)

constexpr int kBlockThreads = 512;       // giant kernels
constexpr int kGiantChunk = 2048;        // edges per giant chunk
constexpr int kGiantCap = 4096;          // slots of a chunk table (2048 edges -> p1 = 4095)
constexpr int kThreadThreads = 256;

thread_local std::string g_err;

int fail(int code, const char *fmt, ...) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    g_err = buf;
    return code;
}

#define CU(call)                                                                             \
    do {                                                                                     \
        cudaError_t e_ = (call);                                                             \
        if (e_ != cudaSuccess)                                                               \
            return fail(e_ == cudaErrorMemoryAllocation ? NULPA_ENOMEM : NULPA_ECUDA,        \
                        "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__,    \
                        __LINE__);                                                           \
    } while (0)

#define CHECK(x)                              \
    do {                                      \
        int r_ = (x);                         \
        if (r_ != NULPA_OK) return r_;        \
    } while (0)

// ---------------------------------------------------------------------------
// device helpers
// ---------------------------------------------------------------------------

// Lemire's fastmod for 32-bit operands: a mod d with M = floor((2^64-1)/d)+1.
__device__ __forceinline__ uint32_t fastmod(uint32_t a, uint64_t M, uint32_t d) {
    uint64_t low = M * a;
    return (uint32_t)__umul64hi(low, d);
}

// R1: capacity p1 = nextPow2(D) - 1 with nextPow2 strictly greater than D;
// R3: p2 = 2*p1 + 1.
__host__ __device__ __forceinline__ uint32_t capacity_p1(uint32_t D) {
#ifdef __CUDA_ARCH__
    return D == 0 ? 0u : (uint32_t)((2ull << (31 - __clz(D))) - 1);
#else
    uint64_t p = 1;
    while (p <= D) p <<= 1;
    return (uint32_t)(p - 1);
#endif
}

// Capacities are Mersenne numbers p = 2^a - 1 (R1, R3), so the fastmod
// magic of every p1 / p2 comes from a compile-time table indexed by a.
struct MagicTable {
    uint64_t m[34];
    constexpr MagicTable() : m() {
        m[0] = 0;
        for (int a = 1; a < 34; ++a) m[a] = UINT64_C(0xFFFFFFFFFFFFFFFF) / ((UINT64_C(1) << a) - 1) + 1;
    }
};
__constant__ MagicTable c_magic = MagicTable();

struct Hash {
    uint32_t p1, p2;
    uint64_t m1, m2;
    __device__ __forceinline__ void init(uint32_t degree) {
        const int a = degree ? 32 - __clz(degree) : 0;   // nextPow2(D) = 2^a (R1)
        p1 = a ? (uint32_t)((UINT64_C(1) << a) - 1) : 0u;
        p2 = 2 * p1 + 1;                                  // R3
        m1 = c_magic.m[a];
        m2 = c_magic.m[a + 1];
    }
};

// Tie order among labels of equal weight (R6, north star): the smallest
// label.  rank(k) maps k to an integer whose order is the tie order
// (identity); kept as a type so the argmax code reads as the rule it applies.
struct TieOrder {
    __device__ __forceinline__ void init(const struct Hash &) {}
    __device__ __forceinline__ uint32_t rank(int32_t k) const { return (uint32_t)k; }
    __device__ __forceinline__ int32_t unrank(uint32_t t) const { return (int32_t)t; }
};

// hashtableAccumulate, Algorithm 2, the SHARED branch:
// atomicCAS claims an empty slot, atomicAdd accumulates.  Works on shared or
// global memory (generic addressing).  i and delta_i are kept reduced mod p1
// (same slots); R5 linear continuation after kMaxRetries probes.
// Returns true if the key newly claimed a slot (*slot_out = slot).
__device__ __forceinline__ bool ht_accumulate(int32_t *Hk, float *Hv, const Hash &h, int32_t k,
                                              float v, uint32_t *slot_out = nullptr, float *total_out = nullptr) {
    const uint32_t p1 = h.p1;
    uint32_t i = fastmod((uint32_t)k, h.m1, p1);
    uint32_t di = p1 > 1 ? 1u : 0u;
    uint32_t km = fastmod((uint32_t)k, h.m2, h.p2);
    if (km >= p1) km -= p1;
    if (km >= p1) km -= p1;
    for (int t = 0; t < kMaxRetries; ++t) {
        int32_t cur = *((volatile int32_t *)&Hk[i]);
        if (cur == k || cur == kEmpty) {
            int32_t old = cur == k ? k : atomicCAS(&Hk[i], kEmpty, k);
            if (old == kEmpty || old == k) {
                const float prev = atomicAdd(&Hv[i], v);
                if (total_out) *total_out = __fadd_rn(prev, v);
                if (slot_out) *slot_out = i;
                return old == kEmpty;
            }
        }
        i += di;
        if (i >= p1) i -= p1;
        di = 2 * di + km;            // < 2p1 + p1
        if (di >= p1) di -= p1;
        if (di >= p1) di -= p1;
    }
    for (uint32_t t = 0; t < p1; ++t) {     // R5
        int32_t cur = *((volatile int32_t *)&Hk[i]);
        if (cur == k || cur == kEmpty) {
            int32_t old = cur == k ? k : atomicCAS(&Hk[i], kEmpty, k);
            if (old == kEmpty || old == k) {
                const float prev = atomicAdd(&Hv[i], v);
                if (total_out) *total_out = __fadd_rn(prev, v);
                if (slot_out) *slot_out = i;
                return old == kEmpty;
            }
        }
        i = i + 1 == p1 ? 0 : i + 1;
    }
    return false;  // unreachable: distinct keys <= D <= p1
}

// Algorithm 2's probe sequence without the value update: find the slot
// holding k or claim an empty one with atomicCAS (R5 linear continuation).
__device__ __forceinline__ uint32_t ht_claim(int32_t *Hk, const Hash &h, int32_t k, bool *fresh = nullptr) {
    const uint32_t p1 = h.p1;
    uint32_t i = fastmod((uint32_t)k, h.m1, p1);
    uint32_t di = p1 > 1 ? 1u : 0u;
    uint32_t km = fastmod((uint32_t)k, h.m2, h.p2);
    if (km >= p1) km -= p1;
    if (km >= p1) km -= p1;
    if (fresh) *fresh = false;
    for (int t = 0; t < kMaxRetries; ++t) {
        int32_t cur = *((volatile int32_t *)&Hk[i]);
        if (cur == k) return i;
        if (cur == kEmpty) {
            int32_t old = atomicCAS(&Hk[i], kEmpty, k);
            if (old == kEmpty && fresh) *fresh = true;
            if (old == kEmpty || old == k) return i;
        }
        i += di;
        if (i >= p1) i -= p1;
        di = 2 * di + km;
        if (di >= p1) di -= p1;
        if (di >= p1) di -= p1;
    }
    for (uint32_t t = 0; t < p1; ++t) {
        int32_t cur = *((volatile int32_t *)&Hk[i]);
        if (cur == k) return i;
        if (cur == kEmpty) {
            int32_t old = atomicCAS(&Hk[i], kEmpty, k);
            if (old == kEmpty && fresh) *fresh = true;
            if (old == kEmpty || old == k) return i;
        }
        i = i + 1 == p1 ? 0 : i + 1;
    }
    return 0;  // unreachable: distinct keys <= D <= p1
}

// Sum of `x` over the lanes of this lane's match_any group `grp`, delivered
// to the group's lowest lane (rank 0): a pairwise tree over the members in
// lane (= CSR) order.  The member d ranks ahead is found by pointer jumping
// (nxt <- nxt[nxt] doubles the distance each step), two shuffles per level.
// maxn (warp-uniform) = largest group size.
__device__ __forceinline__ float group_sum(unsigned grp, float x, unsigned maxn) {
    const int lane = threadIdx.x & 31;
    const unsigned rank = __popc(grp & ((1u << lane) - 1));
    const unsigned above = lane == 31 ? 0u : grp & (0xFFFFFFFEu << lane);
    int nxt = above ? __ffs(above) - 1 : 32;               // member 1 ahead (32 = none)
    for (unsigned d = 1; d < maxn; d <<= 1) {
        const float y = __shfl_sync(0xFFFFFFFFu, x, nxt & 31);
        const int n2 = __shfl_sync(0xFFFFFFFFu, nxt, nxt & 31);
        if ((rank & (2 * d - 1)) == 0 && nxt < 32) x = __fadd_rn(x, y);
        nxt = nxt < 32 ? n2 : 32;                          // member 2d ahead
    }
    return x;
}

// k_warp tables store for label k the tag (k + 1) | (epoch << kbits), where
// kbits = bit length of the number of labels and the epoch counts the
// vertices a warp has folded since its table was last zeroed (1 ..
// 2^(32-kbits) - 1).  A slot whose tag is below epoch << kbits -- zeroed, or
// written for an earlier vertex -- is empty for the current vertex, so
// hashtableClear is a counter increment, and the table is
// zeroed (16-byte stores of the zero register) only when the epoch wraps:
// every 63 vertices at N = 40M (kbits 26); every vertex when N >= 2^30.
__device__ __forceinline__ uint32_t kv_tag(int32_t k, uint32_t epb) { return (uint32_t)k + 1u + epb; }
__device__ __forceinline__ void sts_v4_empty(uint32_t addr) {
    asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(addr), "r"(0u) : "memory");
}

// (weight, tie rank) packed so that an unsigned max gives the largest weight
// and, among equal weights, the label first in tie order (R6; R12: weights
// >= 0 so IEEE bit patterns order like the values).  0 = no candidate.
__device__ __forceinline__ uint64_t pack_cand(float w, int32_t k, const TieOrder &to) {
    return ((uint64_t)__float_as_uint(w) << 32) | (uint64_t)(0xFFFFFFFFu - to.rank(k));
}
__device__ __forceinline__ int32_t cand_label(uint64_t c, const TieOrder &to) {
    return to.unrank(0xFFFFFFFFu - (uint32_t)(c & 0xFFFFFFFFu));
}
__device__ __forceinline__ uint64_t warp_max_u64(uint64_t x) {
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        uint64_t y = __shfl_xor_sync(0xFFFFFFFFu, x, o);
        x = y > x ? y : x;
    }
    return x;
}

// The move rule, PAPER.md:344 (R7: no candidate -> keep the label).
__device__ __forceinline__ bool accept_move(int32_t cstar, int32_t ci, int pickless) {
    return cstar != kEmpty && cstar != ci && (!pickless || cstar <= ci);
}

#ifndef NULPA_STREAM_LOAD
#define NULPA_STREAM_LOAD 2              // 0: ld.global.cs (evict-first); 1: ld.global.nc; 2: plain ld.global
#endif
template <typename T>
__device__ __forceinline__ T ld_stream(const T *p) {
#if NULPA_STREAM_LOAD == 0
    return __ldcs(p);
#elif NULPA_STREAM_LOAD == 1
    return __ldg(p);
#else
    return *p;
#endif
}
// a label gather C[j] (L2 evict_last / evict_normal cache policies on the
// gathers, and evict_first on the CSR streams, measured neutral or slower:
// DESIGN.md experiments)
__device__ __forceinline__ int32_t ld_label(const int32_t *p) { return *p; }

// CSR indices / weights are streamed once per sweep (ld_stream).  Evict-first
// loads (ld.global.cs), meant to keep them from pushing the gathered label
// vector out of L2, measured 2.7% slower than plain loads once the first
// sweep walks long runs of rows (the flag marking re-reads a changed
// vertex's row), so plain loads are the default.
struct SweepArgs {
    const int64_t *__restrict__ offsets;
    const int32_t *__restrict__ indices;
    const float *__restrict__ weights;
    const int32_t *lab_in;     // async: == lab_out
    int32_t *lab_out;
    uint8_t *flag_in;          // async: == flag_out
    uint8_t *flag_out;
    int64_t row_begin;
    int pickless;
    const int32_t *pl_dev;     // device loop (nulpa_run's CUDA graph): Pick-Less flag in device memory, else null
    int first;                 // first sweep after a reset (labels mostly distinct)
    uint32_t kbits;            // bit length of the number of labels (k_warp table tags)
    unsigned long long *ctr;   // kCtr counters of this iteration
};
// this sweep's Pick-Less flag: from the device loop's state, or the host's
__device__ __forceinline__ int sweep_pl(const SweepArgs &a) { return a.pl_dev ? *a.pl_dev : a.pickless; }

// ---------------------------------------------------------------------------
// thread-per-vertex kernel (degree < switch_degree <= 33), PAPER.md:241-243:
// "only a single thread operates on the hashtable.  This eliminates the need
// for atomic operations".  With at most MAXD neighbours the table lives in
// registers: the weight of label lab[k] is the sum over m of w[m] where
// lab[m] == lab[k], taken in CSR order (bit-identical to a sequential
// float32 hashtable accumulation).
// ---------------------------------------------------------------------------
template <bool SYNC, bool W, int MAXD>
__global__ void __launch_bounds__(kThreadThreads) k_thread(SweepArgs a, const int32_t *__restrict__ list,
                                                           int64_t n, bool consec4) {
    // Grid-stride over the bin list, 4 consecutive entries per thread and
    // step: one 16-byte list load and four independent flag loads, then the
    // unprocessed ones are folded.  Late sweeps of a road network are a scan
    // of mostly pruned vertices; one entry per thread and step made every
    // step two dependent round trips (list -> flag) for one entry.
    __shared__ unsigned long long bctr[4];
    if (threadIdx.x < 4) bctr[threadIdx.x] = 0;
    __syncthreads();
    uint32_t n_act = 0, n_ch = 0;
    unsigned long long e_act = 0, e_ch = 0;
    const int pl = sweep_pl(a);
    auto process = [&](int32_t r) {
        const int64_t v = r + a.row_begin;
        const int64_t o = a.offsets[r];
        const uint32_t deg = (uint32_t)(a.offsets[r + 1] - o);
        int32_t lab[MAXD];
        float w[MAXD];
#pragma unroll
        for (int k = 0; k < MAXD; ++k) {
            lab[k] = kEmpty;
            w[k] = 0.0f;
            if (k < (int)deg) {
                const int32_t j = a.indices[o + k];
                if (j != (int32_t)v) {                      // "if j = i continue"
                    lab[k] = a.lab_in[j];
                    w[k] = W ? a.weights[o + k] : 1.0f;
                }
            }
        }
        TieOrder to;
        uint64_t best = 0;
#pragma unroll
        for (int k = 0; k < MAXD; ++k) {
            if (k >= (int)deg) break;
            if (lab[k] == kEmpty) continue;
            float s = 0.0f;
#pragma unroll
            for (int m = 0; m < MAXD; ++m) {
                if (m >= (int)deg) break;
                s = __fadd_rn(s, lab[m] == lab[k] ? w[m] : 0.0f);
            }
            const uint64_t c = pack_cand(s, lab[k], to);
            best = c > best ? c : best;
        }
        const int32_t ci = a.lab_in[v];
        const int32_t cs = best ? cand_label(best, to) : kEmpty;
        n_act += 1;
        e_act += deg;
        if (accept_move(cs, ci, pl)) {
            a.lab_out[v] = cs;
            n_ch += 1;
            e_ch += deg;
            for (uint32_t k = 0; k < deg; ++k) a.flag_out[a.indices[o + k]] = 1;
        }
    };
    // step = 4 consecutive entries per thread (bulk bins: ordered sweep,
    // fewer dependent scan round trips) or 1 (thin bins: all parallelism)
    const int64_t nq = consec4 ? (n + 3) / 4 : n;
    for (int64_t q = (int64_t)blockIdx.x * kThreadThreads + threadIdx.x; q < nq; q += (int64_t)gridDim.x * kThreadThreads) {
        int32_t r[4] = {-1, -1, -1, -1};
        if (!consec4) {
            r[0] = list[q];
        } else if (4 * q + 3 < n) {
            const int4 v4 = *reinterpret_cast<const int4 *>(list + 4 * q);   // the bin list is 16-byte aligned
            r[0] = v4.x; r[1] = v4.y; r[2] = v4.z; r[3] = v4.w;
        } else {
#pragma unroll
            for (int u = 0; u < 4; ++u) r[u] = 4 * q + u < n ? list[4 * q + u] : -1;
        }
        bool act[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) act[u] = r[u] >= 0 && a.flag_in[r[u] + a.row_begin] != 0;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            if (!act[u]) continue;                          // "if not unprocessed(i) continue"
            if (!SYNC) a.flag_in[r[u] + a.row_begin] = 0;   // mark i as processed
            process(r[u]);
        }
    }
    // counters: warp sums, then one set of global atomics per CTA
    n_act = __reduce_add_sync(0xFFFFFFFFu, n_act);
    n_ch = __reduce_add_sync(0xFFFFFFFFu, n_ch);
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        e_act += __shfl_xor_sync(0xFFFFFFFFu, e_act, o);
        e_ch += __shfl_xor_sync(0xFFFFFFFFu, e_ch, o);
    }
    if ((threadIdx.x & 31) == 0 && n_act) {
        atomicAdd(&bctr[0], (unsigned long long)n_act);
        atomicAdd(&bctr[1], e_act);
        atomicAdd(&bctr[2], (unsigned long long)n_ch);
        atomicAdd(&bctr[3], e_ch);
    }
    __syncthreads();
    if (threadIdx.x == 0 && bctr[0]) {
        atomicAdd(&a.ctr[1], bctr[0]);
        atomicAdd(&a.ctr[5], bctr[1]);
        if (bctr[2]) {
            atomicAdd(&a.ctr[0], bctr[2]);
            atomicAdd(&a.ctr[9], bctr[2]);
            atomicAdd(&a.ctr[13], bctr[3]);
        }
    }
}

// ---------------------------------------------------------------------------
// Thread bin over a compacted frontier (asynchronous mode, bulk thread bins:
// road / k-mer graphs, where the thread bin is the whole sweep).  k_tscan is
// the vertex-pruning test of Algorithm 1 as a streaming
// pass over a slice of the bin list: the unprocessed rows, in list order
// within each CTA tile, are appended to `out` and their flags cleared ("mark
// i as processed"); one global atomic per tile.  k_tact then gives every
// thread 4 consecutive compacted rows (the ID-order propagation of the
// grid-stride k_thread: vertex u sees the labels rows u-1.. of its quad
// wrote) and issues the loads of all 4 of them at once -- offsets, indices,
// weights, neighbour labels -- before deciding them in order; a label
// gathered before an earlier row of the quad moved is patched to the new
// label (as k_warp does for its pipelined vertex).  Late sweeps of a road
// network process a few percent of the bin: the plain grid-stride kernel
// pays its dependent list -> flag -> offsets -> indices -> labels round
// trips on every step of every warp; here only the active rows are visited,
// with all their loads in flight.
// ---------------------------------------------------------------------------
constexpr int kTScanThreads = 256;
__global__ void __launch_bounds__(kTScanThreads) k_tscan(SweepArgs a, const int32_t *__restrict__ list, int64_t n,
                                                         int32_t *__restrict__ out, unsigned long long *count) {
    constexpr int NW = kTScanThreads / 32;
    __shared__ uint32_t s_w[NW];
    __shared__ unsigned long long s_base;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int64_t tile = (int64_t)blockIdx.x * kTScanThreads * 4; tile < n; tile += (int64_t)gridDim.x * kTScanThreads * 4) {
        const int64_t q = tile + 4 * (int64_t)threadIdx.x;
        int32_t r[4] = {-1, -1, -1, -1};
        if (q + 3 < n) {
            const int4 v4 = *reinterpret_cast<const int4 *>(list + q);     // slices start on 16-byte boundaries
            r[0] = v4.x; r[1] = v4.y; r[2] = v4.z; r[3] = v4.w;
        } else {
#pragma unroll
            for (int u = 0; u < 4; ++u) r[u] = q + u < n ? list[q + u] : -1;
        }
        bool act[4];
        uint32_t c = 0;
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            act[u] = r[u] >= 0 && a.flag_in[r[u] + a.row_begin] != 0;
            c += act[u];
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (act[u]) a.flag_in[r[u] + a.row_begin] = 0;          // mark i as processed
        uint32_t incl = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(0xFFFFFFFFu, incl, o);
            if (lane >= o) incl += t;
        }
        if (lane == 31) s_w[wid] = incl;
        __syncthreads();
        if (threadIdx.x == 0) {
            uint32_t tot = 0;
#pragma unroll
            for (int w = 0; w < NW; ++w) tot += s_w[w];
            s_base = tot ? atomicAdd(count, (unsigned long long)tot) : 0;
        }
        __syncthreads();
        unsigned long long pos = s_base + incl - c;
        for (int w = 0; w < wid; ++w) pos += s_w[w];
#pragma unroll
        for (int u = 0; u < 4; ++u)
            if (act[u]) out[pos++] = r[u];
        __syncthreads();                                          // s_w / s_base reused by the next tile
    }
}

// V rows of a quad have their loads in flight together (V = 4: road, and
// k-mer at MAXD 8 with NULPA_TACT_V8)
template <bool W, int MAXD, int V>
__global__ void __launch_bounds__(kThreadThreads) k_tact(SweepArgs a, const int32_t *__restrict__ rows,
                                                         const unsigned long long *__restrict__ count) {
    __shared__ unsigned long long bctr[4];
    if (threadIdx.x < 4) bctr[threadIdx.x] = 0;
    __syncthreads();
    const int64_t n = (int64_t)*count;
    uint32_t n_act = 0, n_ch = 0;
    unsigned long long e_act = 0, e_ch = 0;
    const int pl = sweep_pl(a);
    for (int64_t q = (int64_t)blockIdx.x * kThreadThreads + threadIdx.x; 4 * q < n; q += (int64_t)gridDim.x * kThreadThreads) {
#pragma unroll
        for (int h = 0; h < 4; h += V) {
            // rows of this group that moved (-2: did not) and their new labels;
            // earlier groups wrote their labels before this group's loads
            int32_t vmov[V], cmov[V];
            int32_t v[V], ci[V], lab[V][MAXD], jj[V][MAXD];
            float w[V][MAXD];
            int64_t o[V];
            uint32_t deg[V];
#pragma unroll
            for (int u = 0; u < V; ++u) {
                const int64_t e = 4 * q + h + u;
                v[u] = -1;
                deg[u] = 0;
                o[u] = 0;
                ci[u] = 0;
                vmov[u] = -2;
                cmov[u] = 0;
                if (e < n) {
                    const int32_t r = rows[e];
                    v[u] = (int32_t)(r + a.row_begin);
                    o[u] = a.offsets[r];
                    deg[u] = (uint32_t)(a.offsets[r + 1] - o[u]);
                    ci[u] = a.lab_in[v[u]];
                }
            }
#pragma unroll
            for (int u = 0; u < V; ++u)
#pragma unroll
                for (int k = 0; k < MAXD; ++k) {
                    jj[u][k] = -1;
                    lab[u][k] = kEmpty;
                    w[u][k] = 0.0f;
                    if (k < (int)deg[u]) {
                        jj[u][k] = a.indices[o[u] + k];
                        if (W) w[u][k] = a.weights[o[u] + k];
                    }
                }
#pragma unroll
            for (int u = 0; u < V; ++u)
#pragma unroll
                for (int k = 0; k < MAXD; ++k)
                    if (jj[u][k] >= 0 && jj[u][k] != v[u]) {        // "if j = i continue"
                        lab[u][k] = a.lab_in[jj[u][k]];
                        if (!W) w[u][k] = 1.0f;
                    }
#pragma unroll
            for (int u = 0; u < V; ++u) {
                if (v[u] < 0) continue;
                // labels gathered before an earlier row of the group moved
#pragma unroll
                for (int p = 0; p < u; ++p)
#pragma unroll
                    for (int k = 0; k < MAXD; ++k)
                        if (jj[u][k] == vmov[p]) lab[u][k] = cmov[p];
                TieOrder to;
                uint64_t best = 0;
#pragma unroll
                for (int k = 0; k < MAXD; ++k) {
                    if (lab[u][k] == kEmpty) continue;
                    float s = 0.0f;
#pragma unroll
                    for (int m = 0; m < MAXD; ++m) s = __fadd_rn(s, lab[u][m] == lab[u][k] ? w[u][m] : 0.0f);
                    const uint64_t c = pack_cand(s, lab[u][k], to);
                    best = c > best ? c : best;
                }
                const int32_t cs = best ? cand_label(best, to) : kEmpty;
                n_act += 1;
                e_act += deg[u];
                if (accept_move(cs, ci[u], pl)) {
                    a.lab_out[v[u]] = cs;
                    n_ch += 1;
                    e_ch += deg[u];
#pragma unroll
                    for (int k = 0; k < MAXD; ++k)
                        if (jj[u][k] >= 0) a.flag_out[jj[u][k]] = 1;
                    vmov[u] = v[u];
                    cmov[u] = cs;
                }
            }
        }
    }
    n_act = __reduce_add_sync(0xFFFFFFFFu, n_act);
    n_ch = __reduce_add_sync(0xFFFFFFFFu, n_ch);
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        e_act += __shfl_xor_sync(0xFFFFFFFFu, e_act, o);
        e_ch += __shfl_xor_sync(0xFFFFFFFFu, e_ch, o);
    }
    if ((threadIdx.x & 31) == 0 && n_act) {
        atomicAdd(&bctr[0], (unsigned long long)n_act);
        atomicAdd(&bctr[1], e_act);
        atomicAdd(&bctr[2], (unsigned long long)n_ch);
        atomicAdd(&bctr[3], e_ch);
    }
    __syncthreads();
    if (threadIdx.x == 0 && bctr[0]) {
        atomicAdd(&a.ctr[1], bctr[0]);
        atomicAdd(&a.ctr[5], bctr[1]);
        if (bctr[2]) {
            atomicAdd(&a.ctr[0], bctr[2]);
            atomicAdd(&a.ctr[9], bctr[2]);
            atomicAdd(&a.ctr[13], bctr[3]);
        }
    }
}

// ---------------------------------------------------------------------------
// k_warp's per-vertex hashtable: one warp-private table in shared memory,
// reused by every vertex the warp processes.  Capacity by degree class,
// p1 in {255, 511} (a Mersenne number as in R1/R3, load factor <= 1/4 for
// D < 64 and <= 1/2 above; PAPER.md:208 sizes per-vertex GLOBAL tables
// p1 = nextPow2(D)-1 -- the giant bin keeps that sizing).  One 64-bit word
// per slot {tag k+1, float value}, so a probe is ONE ld.shared.v2 and an
// empty slot is all-zero (its value 0.0f, so "claim" and "hit" both store
// old value + x); the table is cleared with 16-byte stores of the zero
// register before each vertex (hashtableClear).  Keys within
// one 32-entry batch are distinct (one leader per label, match_any) and
// batches are ordered by __syncwarp, so the value update is a plain
// read-modify-write; only the slot claim is atomic.
// ---------------------------------------------------------------------------
constexpr int kWarpSlots = 512;          // largest class: p1 = 511

// Slot claims without atomics.  A full-warp shared-memory atomic costs ~2
// cycles per active lane of the SM's atomics unit (B300_MICROARCH.md
// "Atomics"), and in the first sweep ~25 leaders per batch claim new slots,
// so the claim is a warp-synchronous round instead: every probing lane
// reads its slot (one ld.shared.v2 per lane), lanes that find their tag are
// done (hit), lanes that find it empty store their tag, __syncwarp, and
// re-read it -- of several lanes storing to one slot in the same round
// exactly one store survives, that lane won the claim, the others probe on.
// The value update is old value + x (an empty slot holds 0.0f), stored by
// the lane that owns the label's slot.  `need` lanes probe; on return they
// are done (need = false) or collided.
// Every lane reads (lanes that do not probe read the slot of their own
// group's key -- the leader's address -- or of kEmpty, so the read is a
// broadcast and costs no extra wavefront; no default values to set up).
// NULPA_WARP_SYNC 0 drops the bar.warp.sync between the claim store and the
// re-read: the warp is converged here (every caller is warp-synchronous
// code with full-mask votes) and its shared-memory instructions complete in
// order, and every re-reading lane stored to that address itself.
#ifndef NULPA_WARP_SYNC
#define NULPA_WARP_SYNC 1
#endif
#ifndef NULPA_BLOCK_LIST
#define NULPA_BLOCK_LIST 1               // k_block: list the claimed slots; scan and reset only those
#endif
#ifndef NULPA_MAJORITY
#define NULPA_MAJORITY 1                 // k_warp, k_block, giant bin: strict-majority shortcut for the vertex's own label (not the first sweep)
#endif
#ifndef NULPA_EPOCH
#define NULPA_EPOCH 1                    // 0: zero the k_warp table before every vertex
#endif
#if NULPA_WARP_SYNC
#define KV_WSYNC "bar.warp.sync 0xFFFFFFFF;\n\t"
__device__ __forceinline__ void wsync() { __syncwarp(); }
#else
#define KV_WSYNC ""
__device__ __forceinline__ void wsync() { asm volatile("" ::: "memory"); }
#endif
__device__ __forceinline__ void kv_round(uint32_t addr, uint32_t tg, uint32_t epb, float x, bool &need, float &V) {
    uint32_t n = need, vb = __float_as_uint(V);
    asm volatile(
        "{\n\t"
        ".reg .pred pn, ph, pc, pd;\n\t"
        ".reg .b32 ck, now;\n\t"
        ".reg .f32 cv, nv;\n\t"
        "setp.ne.b32 pn, %0, 0;\n\t"
        "ld.shared.v2.b32 {ck, cv}, [%2];\n\t"
        "setp.eq.and.b32 ph, ck, %3, pn;\n\t"      // the label's slot: hit
        "setp.lt.and.u32 pc, ck, %5, pn;\n\t"      // empty (zeroed or an earlier vertex's): try to claim
        "@pc st.shared.b32 [%2], %3;\n\t"
        KV_WSYNC
        "@pc ld.shared.b32 now, [%2];\n\t"
        "setp.eq.and.b32 pd, now, %3, pc;\n\t"     // this lane's store survived: claimed
        "@!ph mov.f32 cv, 0f00000000;\n\t"         // a claimed slot starts at 0
        "or.pred pd, pd, ph;\n\t"
        "add.rn.f32 nv, cv, %4;\n\t"
        "@pd st.shared.f32 [%2+4], nv;\n\t"
        "@pd mov.b32 %1, nv;\n\t"
        "@pd mov.b32 %0, 0;\n\t"
        "}"
        : "+r"(n), "+r"(vb)
        : "r"(addr), "r"(tg), "f"(x), "r"(epb)
        : "memory");
    need = n != 0;
    V = __uint_as_float(vb);
}

// Algorithm 2's probe sequence past probe 1 (home + 1; the step delta_0 = 1
// has become delta_1 = 2 + (k mod p2) mod P): hybrid quadratic-double
// probing, R5 linear continuation after kMaxRetries probes.  Called by the
// whole warp (rounds are warp-synchronous); lanes without `need` idle.
template <uint32_t P>
__device__ __noinline__ float kv_add_slow(uint32_t tab, int32_t k, uint32_t epb, float x, uint32_t i, bool need, float V) {
    constexpr uint32_t p2 = 2 * P + 1;                    // R3
    const uint32_t km = ((uint32_t)k % p2) % P;
    uint32_t di = 2 + km;
    if (di >= P) di -= P;
    const uint32_t tg = kv_tag(k, epb);
    for (int t = 2; __any_sync(0xFFFFFFFFu, need); ++t) {
        if (t <= kMaxRetries) {
            i += di;
            if (i >= P) i -= P;
            di = 2 * di + km;
            if (di >= P) di -= P;
            if (di >= P) di -= P;
        } else {
            i = i + 1 == P ? 0 : i + 1;                    // R5
        }
        kv_round(tab + 8 * i, tg, epb, x, need, V);
    }
    return V;
}

// hashtableAccumulate (Algorithm 2) by the group leaders of one batch (`on`),
// adding group weight x to label k: the home slot k mod P and probe 1
// (home + 1) inline, later probes out of line.  Returns the label's new
// total (leaders only).  Warp-synchronous: called by all 32 lanes.
template <uint32_t P>
__device__ __forceinline__ float kv_add(uint32_t tab, int32_t k, uint32_t epb, float x, bool on) {
    const uint32_t tg = kv_tag(k, epb);
    const uint32_t i0 = (uint32_t)k % P;
    float V = 0.0f;
    bool need = on;
    kv_round(tab + 8 * i0, tg, epb, x, need, V);
    if (__any_sync(0xFFFFFFFFu, need)) {
        const uint32_t i1 = i0 + 1 == P ? 0u : i0 + 1;
        kv_round(tab + 8 * i1, tg, epb, x, need, V);
        if (__any_sync(0xFFFFFFFFu, need)) V = kv_add_slow<P>(tab, k, epb, x, i1, need, V);
    }
    return V;
}

// ---------------------------------------------------------------------------
// Frontier compaction (vertex pruning, "if not unprocessed(i)
// continue; mark i as processed"): one pass over a bin list writes a 16-byte
// record {offset, degree, row, C[i]} per unprocessed vertex and clears its
// flag (async).  The warp kernel then streams records at known addresses, so
// the loads of upcoming vertices can be issued ahead (software pipelining)
// instead of waiting on list -> flag -> offsets dependent round trips.
// C[i] read here is still C[i] when i is processed: only i writes C[i].
// Also counts processed vertices and their edges (counters 1+bin, 5+bin).
// ---------------------------------------------------------------------------
struct __align__(16) VRec {
    uint32_t o_lo;      // offsets[r], low 32 bits
    uint32_t o_hi_deg;  // offsets[r] bits 32..47 | degree << 16 (degree < 2^16 in the warp bin)
    int32_t r;          // local row
    int32_t ci;         // C[i]
};

// With a split degree (block bin): records of degree < split go to recs
// (count), the others to recs2 (count2).  Positions are reserved with ONE
// global atomic per CTA tile of kFrontTile list entries (a single counter
// hit by one atomic per warp serialised ~1M atomics at L2: ~1 ms per sweep);
// within a tile, records keep list (row) order.
#ifndef NULPA_FRONT_PER
#define NULPA_FRONT_PER 1
#endif
constexpr int kFrontThreads = 256, kFrontPer = NULPA_FRONT_PER, kFrontTile = kFrontThreads * kFrontPer;
template <bool SYNC>
__global__ void __launch_bounds__(kFrontThreads) k_frontier(SweepArgs a, const int32_t *__restrict__ list, int64_t n,
                                                           int bin, VRec *__restrict__ recs,
                                                           unsigned long long *count, uint32_t split,
                                                           VRec *__restrict__ recs2, unsigned long long *count2) {
    constexpr int NW = kFrontThreads / 32;
    __shared__ uint32_t s_c[2][NW];
    __shared__ unsigned long long s_base[2];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint32_t c_act = 0;
    unsigned long long c_edges = 0;
    for (int64_t tile = (int64_t)blockIdx.x * kFrontTile; tile < n; tile += (int64_t)gridDim.x * kFrontTile) {
        // warp w owns entries tile + w*32*kFrontPer + [0, 32*kFrontPer), in 32-entry rounds
        VRec rec[kFrontPer];
        unsigned m[kFrontPer], m2[kFrontPer];
        uint32_t c1 = 0, c2 = 0;
#pragma unroll
        for (int k = 0; k < kFrontPer; ++k) {
            const int64_t t = tile + (wid * kFrontPer + k) * 32 + lane;
            int f = 0;
            uint32_t deg = 0;
            if (t < n) {
                const int32_t r = list[t];
                const int64_t v = r + a.row_begin;
                f = a.flag_in[v];
                if (f) {
                    const int64_t o = a.offsets[r];
                    deg = (uint32_t)(a.offsets[r + 1] - o);
                    rec[k].o_lo = (uint32_t)o;
                    rec[k].o_hi_deg = (uint32_t)((uint64_t)o >> 32) | (deg << 16);
                    rec[k].r = r;
                    rec[k].ci = a.lab_in[v];
                    if (!SYNC) a.flag_in[v] = 0;          // mark i as processed
                }
            }
            const bool hi = f && deg >= split;
            m[k] = __ballot_sync(0xFFFFFFFFu, f && !hi);
            m2[k] = __ballot_sync(0xFFFFFFFFu, hi);
            c1 += __popc(m[k]);
            c2 += __popc(m2[k]);
            c_edges += __reduce_add_sync(0xFFFFFFFFu, deg);
        }
        c_act += c1 + c2;
        if (lane == 0) {
            s_c[0][wid] = c1;
            s_c[1][wid] = c2;
        }
        __syncthreads();
        if (threadIdx.x < 2) {
            uint32_t tot = 0;
#pragma unroll
            for (int w = 0; w < NW; ++w) tot += s_c[threadIdx.x][w];
            s_base[threadIdx.x] = tot ? atomicAdd(threadIdx.x ? count2 : count, (unsigned long long)tot) : 0;
        }
        __syncthreads();
        unsigned long long p1 = s_base[0], p2 = s_base[1];
        for (int w = 0; w < wid; ++w) {
            p1 += s_c[0][w];
            p2 += s_c[1][w];
        }
        __syncthreads();                                  // s_c / s_base reused by the next tile
#pragma unroll
        for (int k = 0; k < kFrontPer; ++k) {
            const unsigned below = (1u << lane) - 1;
            if (m[k] >> lane & 1) recs[p1 + __popc(m[k] & below)] = rec[k];
            if (m2[k] >> lane & 1) recs2[p2 + __popc(m2[k] & below)] = rec[k];
            p1 += __popc(m[k]);
            p2 += __popc(m2[k]);
        }
    }
    __shared__ unsigned long long bctr[2];
    if (threadIdx.x < 2) bctr[threadIdx.x] = 0;
    __syncthreads();
    if (lane == 0 && c_act) {
        atomicAdd(&bctr[0], (unsigned long long)c_act);
        atomicAdd(&bctr[1], c_edges);
    }
    __syncthreads();
    if (threadIdx.x == 0 && bctr[0]) {
        atomicAdd(&a.ctr[1 + bin], bctr[0]);
        atomicAdd(&a.ctr[5 + bin], bctr[1]);
    }
}

// ---------------------------------------------------------------------------
// warp-per-vertex kernel (switch_degree <= D < block_degree; the wide variant
// serves the block bin below wide_degree), over the compacted frontier and
// software-pipelined across the vertices of a warp.  A warp walks its record
// groups (32 records each; 4 in the wide variant) as one sequence
// n = 0, 1, ...; while vertex n is folded, the label gathers of vertex n+1
// and the index/weight loads of vertex n+2 are in flight, so each dependent
// global round trip overlaps a whole vertex of work.  Records reach shared
// memory one group ahead (a 2-group ring per warp).
// Per 32-entry batch: match_any folds lanes holding the same label onto a
// leader, whose group total (count * w when the vertex's weights are all
// equal, else a pairwise tree) is added into the table (Algorithm 2); each
// lane keeps the best (total, label) it produced as a leader, and a
// redux.max / redux.min pair gives hashtableMaxKey without scanning the
// table (ties: smallest label, R6).  Degree <= 32 needs no table (the match
// groups are the totals).
// Asynchronous reading: vertex n+1's neighbour labels are gathered before
// vertex n's new label is written; the gathered copies of that label are
// patched in registers, so n+1 still sees n's move.
//
// Which record groups a warp walks (WarpSched):
//  * SCHED_STEAL (first sweep after a reset): warp w owns the contiguous
//    groups [w*ng/nw, (w+1)*ng/nw) -- one long run of consecutive rows, so
//    labels propagate along ID order as in the sequential Algorithm 1
//    (modularity) -- and a warp that runs dry
//    steals the far half of the remaining range of the most-loaded of 32
//    sampled warps (the victim's run continues undisturbed; the tail is
//    balanced).  A range is one 64-bit word {next group, end group}: the
//    owner takes a group with atomicAdd on the low half, a thief shrinks
//    the high half with atomicCAS.
//  * SCHED_GUIDED (K > 1): guided chunks of min(K, groups left / nw)
//    consecutive groups from a global counter.
//  * SCHED_STRIDED (K = 1): groups w, w + nw, ...
// ---------------------------------------------------------------------------
#ifndef NULPA_WARP_WARPS
#define NULPA_WARP_WARPS 8
#endif
constexpr int kWarpWarps = NULPA_WARP_WARPS;   // warps per CTA
#ifndef NULPA_WARP_CTAS
#define NULPA_WARP_CTAS 4
#endif
constexpr int kWarpCtasPerSm = NULPA_WARP_CTAS;   // 32 warps/SM
// The wide variant (block-bin vertices below wide_degree <= 1024): 1024-slot
// tables (8 KB per warp, p1 = 1023), 4 warps per CTA, 6 CTAs (24 warps) per SM.
constexpr int kWideSlots = 1024, kWideWarps = 4, kWideCtasPerSm = 6;
#ifndef NULPA_WIDE_GROUP
#define NULPA_WIDE_GROUP 4
#endif
#ifndef NULPA_T255_MAX
#define NULPA_T255_MAX 33                // k_warp: 255-slot tables below this degree, 511 above (33: always 511 -- with epoch tags a bigger table costs no clearing and has fewer collisions: web 72.5 -> 73.9e9 edges/s)
#endif
#ifndef NULPA_FIRST_BIG
#define NULPA_FIRST_BIG 0                // 1: 511-slot tables for every degree in the first sweep
#endif
#ifndef NULPA_WIDE_TMA
#define NULPA_WIDE_TMA 1                 // block bin below wide_degree: TMA k_block (128 threads) instead of the wide k_warp
#endif
#ifndef NULPA_WIDE_K
#define NULPA_WIDE_K 2                   // wide schedule: guided chunks of <= this many groups
#endif
template <int SLOTS> struct WarpCfg {
    static constexpr int warps = SLOTS == kWarpSlots ? kWarpWarps : kWideWarps;
    static constexpr int ctas = SLOTS == kWarpSlots ? kWarpCtasPerSm : kWideCtasPerSm;
    static constexpr int unroll = SLOTS == kWarpSlots ? 2 : 4;   // 32-entry batches per loop step past 64
    static constexpr int group = SLOTS == kWarpSlots ? 32 : NULPA_WIDE_GROUP;
};

enum { SCHED_STRIDED = 0, SCHED_GUIDED = 1, SCHED_STEAL = 2 };
#ifndef NULPA_MIN_RUN
#define NULPA_MIN_RUN 2048
#endif
constexpr int64_t kMinFirstRun = NULPA_MIN_RUN;   // rows per warp in the first sweep, at least (small bins)
constexpr double kLocalRuns = 0.5;                // ... if >= this share of the sampled CSR entries are near (k_locality)
struct WarpSched {
    int mode;
    int K;                               // guided chunk size (groups)
    unsigned long long *counter;         // guided: next group
    unsigned long long *ranges;          // steal: one {next, end} word per warp
};

// The warp's next record group, or 0xFFFFFFFF once the warp's share of the
// frontier is exhausted (sticky).  Warp-uniform.
struct GroupFetcher {
    uint32_t cur, lim;                   // strided: next group; guided: chunk [cur, lim)
    uint32_t ng, nw, gw;
    bool dry;
    __device__ __forceinline__ uint32_t next(const WarpSched &s, int lane) {
        if (dry) return 0xFFFFFFFFu;
        uint32_t g = 0xFFFFFFFFu;
        if (s.mode == SCHED_STRIDED) {
            if (cur < ng) g = cur;
            cur += nw;
        } else if (s.mode == SCHED_GUIDED) {
            if (cur >= lim) {
                uint32_t start = 0, size = 1;
                if (lane == 0) {
                    const uint32_t done = (uint32_t)min((unsigned long long)ng, *(volatile unsigned long long *)s.counter);
                    size = max(1u, min((uint32_t)s.K, (ng - done) / nw));
                    start = (uint32_t)min((unsigned long long)ng, atomicAdd(s.counter, (unsigned long long)size));
                }
                cur = __shfl_sync(0xFFFFFFFFu, start, 0);
                lim = min(ng, cur + __shfl_sync(0xFFFFFFFFu, size, 0));
            }
            if (cur < lim) g = cur++;
        } else {                                           // SCHED_STEAL
            for (;;) {
                if (lane == 0) {
                    const unsigned long long w = atomicAdd(s.ranges + gw, 1ull);   // next group of the own range
                    g = (uint32_t)w < (uint32_t)(w >> 32) ? (uint32_t)w : 0xFFFFFFFFu;
                }
                g = __shfl_sync(0xFFFFFFFFu, g, 0);
                if (g != 0xFFFFFFFFu || !steal(s, lane)) break;
            }
        }
        dry = g == 0xFFFFFFFFu;
        return g;
    }
    // Sample 32 warps per round (one per lane), pick the one with the most
    // groups left and move the far half of its range into the own word.
    // false after 8 rounds without a warp holding >= 2 groups.
    __device__ __noinline__ bool steal(const WarpSched &s, int lane) {
        int fails = 0;
        for (uint32_t round = 0; round < 8;) {
            uint32_t h = (gw * 0x9E3779B9u) ^ ((round * 32u + (uint32_t)lane + 1u) * 0x85EBCA6Bu);
            h ^= h >> 15;
            h *= 0x2C1B3C6Du;
            h ^= h >> 12;
            const uint32_t v = h % nw;
            unsigned long long w = 0;
            int32_t rem = 0;
            if (v != gw) {
                w = *(volatile unsigned long long *)(s.ranges + v);
                rem = (int32_t)((uint32_t)(w >> 32) - (uint32_t)w);
            }
            const int32_t best = __reduce_max_sync(0xFFFFFFFFu, rem);
            if (best < 2) {
                ++round;
                continue;
            }
            const int src = __ffs(__ballot_sync(0xFFFFFFFFu, rem == best)) - 1;
            uint32_t ok = 0;
            if (lane == src) {
                const uint32_t lo = (uint32_t)w, hi = (uint32_t)(w >> 32);
                const uint32_t mid = hi - (uint32_t)rem / 2;           // victim keeps [lo, mid)
                if (atomicCAS(s.ranges + v, w, ((unsigned long long)mid << 32) | lo) == w) {
                    atomicExch(s.ranges + gw, ((unsigned long long)hi << 32) | mid);
                    ok = 1;
                }
            }
            if (__shfl_sync(0xFFFFFFFFu, ok, src)) return true;
            if (++fails > 32) return false;                // lost races: try the same round again
        }
        return false;
    }
};

// The fold of one vertex by one warp (lines 337-343 of Algorithm 1): the
// first 64 row entries arrive as labels k0a / k0b (entries lane, lane + 32;
// kEmpty = absent or the vertex itself) with weights w0a / w0b, later entries
// are loaded here.  Returns hashtableMaxKey (kEmpty if no neighbour).
template <bool W, int SLOTS, bool O32>
__device__ __forceinline__ int32_t warp_fold(const SweepArgs &a, uint32_t tab, int lane, unsigned lanes_below,
                                             uint64_t row_o, uint32_t dk, int32_t vk, int32_t ci, int32_t k0a,
                                             int32_t k0b, float w0a, float w0b, uint32_t &ep) {
    constexpr int U = WarpCfg<SLOTS>::unroll;
    (void)U;
    const int32_t *__restrict__ lab_in = a.lab_in;
    auto at = [&](uint64_t o, uint32_t k) -> uint64_t { return O32 ? (uint64_t)((uint32_t)o + k) : o + k; };
    uint32_t bw = 0;                                       // best (weight bits + 1) this lane led; 0 = none
    int32_t bk = 0;
    // unit weights stored (the paper's default weight 1) in the first 64
    // entries?  Then a group's total is its size (exact); else a
    // pairwise tree over the group's weights
    bool eqw = true;
    if (W) eqw = __all_sync(0xFFFFFFFFu, (k0a == kEmpty || w0a == 1.0f) && (k0b == kEmpty || w0b == 1.0f));
    auto group_total = [&](unsigned grp, int32_t key, float w, bool eq) -> float {
        if (!W || eq) return (float)__popc(grp);
        const unsigned maxn = __reduce_max_sync(0xFFFFFFFFu, key != kEmpty ? (unsigned)__popc(grp) : 1u);
        return maxn > 1 ? group_sum(grp, w, maxn) : w;
    };
    if (dk <= 32) {
#if NULPA_MAJORITY
        if (!a.first && eqw && 2 * __popc(__ballot_sync(0xFFFFFFFFu, k0a == ci)) > __popc(__ballot_sync(0xFFFFFFFFu, k0a != kEmpty)))
            return ci;                                     // strict majority of the own label (below)
#endif
        const unsigned grp = __match_any_sync(0xFFFFFFFFu, k0a);
        const bool leader = k0a != kEmpty && (grp & lanes_below) == 0;
        const float x = group_total(grp, k0a, w0a, eqw);
        bw = leader ? __float_as_uint(x) + 1 : 0u;
        bk = k0a;
    } else {
#if NULPA_MAJORITY
        // Past the first sweep most neighbourhoods hold one label.  If the
        // vertex's own label C[i] has a strict majority of its (unit)
        // neighbour weights, it is hashtableMaxKey -- no other label can
        // reach its total, so no tie either -- and the vertex does not move:
        // the same decision as the table fold, for two ballots per batch.
        if (!a.first && eqw) {
            uint32_t own = __popc(__ballot_sync(0xFFFFFFFFu, k0a == ci)) + __popc(__ballot_sync(0xFFFFFFFFu, k0b == ci));
            uint32_t tot = __popc(__ballot_sync(0xFFFFFFFFu, k0a != kEmpty)) + __popc(__ballot_sync(0xFFFFFFFFu, k0b != kEmpty));
            if (2 * own > tot) {
                // rows past 64 entries: a majority in the first 64 -- count the
                // rest (two batches of loads in flight per step); on failure the
                // table fold below re-reads them
                bool unit = true;
                const uint64_t el = at(row_o, (uint32_t)lane);
                for (uint32_t b = 64; b < dk && unit; b += 64) {
                    const bool oka = b + lane < dk, okb = b + 32 + lane < dk;
                    const int32_t ja = oka ? ld_stream(a.indices + el + b) : -1;
                    const int32_t jb = okb ? ld_stream(a.indices + el + b + 32) : -1;
                    float xa = 1.0f, xb = 1.0f;
                    if (W && oka) xa = ld_stream(a.weights + el + b);
                    if (W && okb) xb = ld_stream(a.weights + el + b + 32);
                    const int32_t ka = (ja >= 0 && ja != vk) ? ld_label(lab_in + ja) : kEmpty;
                    const int32_t kb = (jb >= 0 && jb != vk) ? ld_label(lab_in + jb) : kEmpty;
                    if (W) unit = __all_sync(0xFFFFFFFFu, (ka == kEmpty || xa == 1.0f) && (kb == kEmpty || xb == 1.0f));
                    own += __popc(__ballot_sync(0xFFFFFFFFu, ka == ci)) + __popc(__ballot_sync(0xFFFFFFFFu, kb == ci));
                    tot += __popc(__ballot_sync(0xFFFFFFFFu, ka != kEmpty)) + __popc(__ballot_sync(0xFFFFFFFFu, kb != kEmpty));
                }
                if (unit && 2 * own > tot) return ci;
            }
        }
#endif
        auto table_row = [&](auto cap) {
            constexpr uint32_t P = decltype(cap)::value;
            // hashtableClear: next epoch; zero the whole table when the epoch wraps
            const uint32_t emax = NULPA_EPOCH ? (1u << (32 - a.kbits)) - 1u : 1u;
            if (++ep > emax) {
#pragma unroll
                for (uint32_t q = 0; q < SLOTS / 64; ++q) sts_v4_empty(tab + 16 * (q * 32 + lane));
                wsync();
                ep = 1;
            }
            const uint32_t epb = ep << a.kbits;
            auto batch = [&](int32_t key, float w, bool eq) {
                const unsigned grp = __match_any_sync(0xFFFFFFFFu, key);
                const bool leader = key != kEmpty && (grp & lanes_below) == 0;
                const float x = group_total(grp, key, w, eq);
                const float V = kv_add<P>(tab, key, epb, x, leader);
                // running best (total, smallest label) as one 64-bit max
                const uint64_t c = ((uint64_t)(__float_as_uint(V) + 1) << 32) | (uint32_t)~key;
                const uint64_t b = ((uint64_t)bw << 32) | (uint32_t)~bk;
                if (leader && c > b) {
                    bw = (uint32_t)(c >> 32);
                    bk = key;
                }
                wsync();
            };
            batch(k0a, w0a, eqw);
            batch(k0b, w0b, eqw);
            const uint64_t el = at(row_o, (uint32_t)lane);
            const int32_t *pi = a.indices + el;
            const float *pw = W ? a.weights + el : nullptr;
            for (uint32_t b = 64; b < dk; b += 32 * U) {
                // U batches per step: all index loads, then all label gathers in flight
                int32_t iu[U], qu[U];
                float xu[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const bool ok = b + 32 * u + lane < dk;
                    iu[u] = ok ? ld_stream(pi + b + 32 * u) : -1;
                    xu[u] = 1.0f;
                    if (W && ok) xu[u] = ld_stream(pw + b + 32 * u);
                }
#pragma unroll
                for (int u = 0; u < U; ++u) qu[u] = (iu[u] >= 0 && iu[u] != vk) ? ld_label(lab_in + iu[u]) : kEmpty;
                bool eq = true;
                if (W) {
                    bool e = true;
#pragma unroll
                    for (int u = 0; u < U; ++u) e = e && (qu[u] == kEmpty || xu[u] == 1.0f);
                    eq = __all_sync(0xFFFFFFFFu, e);
                }
#pragma unroll
                for (int u = 0; u < U; ++u)
                    if (u == 0 || b + 32 * u < dk) batch(qu[u], xu[u], eq);
            }
        };
        if constexpr (SLOTS == kWideSlots) {
            table_row(std::integral_constant<uint32_t, kWideSlots - 1>());
        } else {
            if (dk < NULPA_T255_MAX && !(NULPA_FIRST_BIG && a.first)) table_row(std::integral_constant<uint32_t, 255>());
            else table_row(std::integral_constant<uint32_t, 511>());
        }
    }
    // hashtableMaxKey: the largest total, ties to the smallest label (R6)
    const uint32_t W1 = __reduce_max_sync(0xFFFFFFFFu, bw);
    const int32_t cs = W1 ? (int32_t)__reduce_min_sync(0xFFFFFFFFu, bw == W1 ? (uint32_t)bk : 0xFFFFFFFFu) : kEmpty;
    return cs;
}

// O32: every CSR offset + 64 fits 32 bits (M < 2^32 - 64): row addresses
// are one 32-bit add + IMAD.WIDE instead of 48-bit arithmetic.
template <bool SYNC, bool W, int SLOTS, bool O32>
__global__ void __launch_bounds__(WarpCfg<SLOTS>::warps * 32, WarpCfg<SLOTS>::ctas)
    k_warp(SweepArgs a, const VRec *__restrict__ recs, const unsigned long long *__restrict__ count, int bin,
           WarpSched ws) {
    constexpr int NWARP = WarpCfg<SLOTS>::warps;
    constexpr int G = WarpCfg<SLOTS>::group;
    constexpr uint32_t RING = 2 * G;
    static_assert(G >= 1 && G <= 32 && (G & (G - 1)) == 0, "group size: power of two <= 32");
    __shared__ __align__(16) uint64_t s_tab[NWARP][SLOTS];
    // two groups; record m sits at m mod 2G, and records 0, 1 again at 2G,
    // 2G+1 (so records n+1, n+2 are at fixed offsets from record n)
    __shared__ __align__(16) VRec s_ring[NWARP][RING + 2];
    __shared__ unsigned long long bctr[2];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const uint32_t tab = (uint32_t)__cvta_generic_to_shared(&s_tab[wid][0]);
    const uint32_t ring = (uint32_t)__cvta_generic_to_shared(&s_ring[wid][0]);
    const unsigned lanes_below = (1u << lane) - 1;
    if (threadIdx.x < 2) bctr[threadIdx.x] = 0;
    const uint32_t nrec = (uint32_t)*count;
    const int pl = sweep_pl(a);
    GroupFetcher F;
    F.ng = (nrec + G - 1) / G;
    F.nw = gridDim.x * NWARP;
    F.gw = blockIdx.x * NWARP + wid;
    F.cur = ws.mode == SCHED_STRIDED ? F.gw : 0;
    F.lim = 0;
    F.dry = false;
    if (ws.mode == SCHED_STEAL && lane == 0) {
        // initial ranges of >= K groups each (K = kMinFirstRun / 32: long runs
        // on small bins); warps past ng / K start empty and only steal
        const uint32_t nr = max(1u, min(F.nw, F.ng / max(1, ws.K)));
        const uint32_t b = F.gw < nr ? (uint32_t)((uint64_t)F.gw * F.ng / nr) : 0u;
        const uint32_t e = F.gw < nr ? (uint32_t)((uint64_t)(F.gw + 1) * F.ng / nr) : 0u;
        atomicExch(ws.ranges + F.gw, ((unsigned long long)e << 32) | b);
    }
    __syncthreads();
    // lane's record of group g.  Past the warp's last group: end records
    // (r = -1); past the bin inside the bin's last group: degree-0 no-op
    // records (with work stealing the bin's last group need not be the
    // warp's last)
    auto grec = [&](uint32_t g) -> VRec {
        if (g == 0xFFFFFFFFu || lane >= G) return VRec{0, 0, -1, 0};
        const uint32_t i = g * G + lane;
        return i < nrec ? recs[i] : VRec{0, 0, 0, 0};
    };
    auto rrec_at = [&](uint32_t addr) -> VRec {
        VRec r;
        asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];"
                     : "=r"(r.o_lo), "=r"(r.o_hi_deg), "=r"(r.r), "=r"(r.ci)
                     : "r"(addr) : "memory");
        return r;
    };
    // row offset (48 bit; 32 bit under O32) and degree of a record
    auto r_o = [](const VRec &r) -> uint64_t {
        return O32 ? (uint64_t)r.o_lo : ((uint64_t)(r.o_hi_deg & 0xFFFFu) << 32) | r.o_lo;
    };
    auto r_d = [](const VRec &r) -> uint32_t { return r.o_hi_deg >> 16; };
    // group -> ring slots [base, base + G) (+ the copy of records 0, 1)
    auto ring_put = [&](uint32_t base, const VRec &r) {
        if (lane < G) s_ring[wid][base + lane] = r;
        if (base == 0 && lane < 2) s_ring[wid][RING + lane] = r;
    };
    {
        const VRec r0 = grec(F.next(ws, lane));
        const VRec r1 = grec(F.next(ws, lane));
        ring_put(0, r0);
        ring_put(G, r1);
    }
    VRec pend = grec(F.next(ws, lane));
    wsync();
    const int32_t *__restrict__ lab_in = a.lab_in;
    // row loads: entries lane and lane+32 of the row of record m
    // entry e of the CSR arrays (e = row offset + position)
    auto at = [&](uint64_t o, uint32_t k) -> uint64_t { return O32 ? (uint64_t)((uint32_t)o + k) : o + k; };
    auto load_idx = [&](const VRec &r, int32_t &ja, int32_t &jb) {
        const uint32_t d = r_d(r);
        const int32_t *pi = a.indices + at(r_o(r), (uint32_t)lane);
        ja = (uint32_t)lane < d ? ld_stream(pi) : -1;
        jb = (uint32_t)lane + 32 < d ? ld_stream(pi + 32) : -1;
    };
    auto load_w = [&](const VRec &r, float &wa, float &wb) {
        wa = wb = 1.0f;
        if (W) {
            const uint32_t d = r_d(r);
            const float *pw = a.weights + at(r_o(r), (uint32_t)lane);
            if ((uint32_t)lane < d) wa = ld_stream(pw);
            if ((uint32_t)lane + 32 < d) wb = ld_stream(pw + 32);
        }
    };
    // label gathers ("if j = i continue": the vertex's own entries are skipped)
    auto gather = [&](int32_t vk, int32_t ja, int32_t jb, int32_t &ka, int32_t &kb) {
        ka = (ja >= 0 && ja != vk) ? ld_label(lab_in + ja) : kEmpty;
        kb = (jb >= 0 && jb != vk) ? ld_label(lab_in + jb) : kEmpty;
    };
    // pipeline registers: vertex n (fold) / n+1 (gathers and weight loads in
    // flight) / n+2 (index loads in flight)
    int32_t j0a, j0b, k0a, k0b, j1a, j1b, k1a, k1b, j2a, j2b;
    float w0a, w0b, w1a, w1b;
    {
        load_idx(rrec_at(ring), j0a, j0b);
        load_idx(rrec_at(ring + 16), j1a, j1b);
        load_w(rrec_at(ring), w0a, w0b);
        gather(rrec_at(ring).r + (int32_t)a.row_begin, j0a, j0b, k0a, k0b);
    }
    uint32_t c_ch = 0, c_che = 0;
    uint32_t ep = 0xFFFFFFFEu;                             // table epoch: the first table vertex zeroes the table
    for (uint32_t q = 0;; ++q) {                           // record groups
      if (q > 0) {
          // entering group q (groups q-1, q in the ring): group q+1 (pend)
          // goes where group q-1 was, group q+2 is requested
          ring_put(((q + 1) & 1) * G, pend);
          pend = grec(F.next(ws, lane));
          wsync();
      }
      const uint32_t ring_q = ring + 16u * ((q & 1) * G);
      for (uint32_t p = 0; p < (uint32_t)G; ++p) {          // vertex n = q*G + p
        const uint32_t rn = ring_q + 16u * p;
        const VRec rc = rrec_at(rn);
        if (rc.r < 0) goto done;                           // end record
        const uint32_t dk = r_d(rc);
        load_idx(rrec_at(rn + 32), j2a, j2b);
        {
            const VRec r1 = rrec_at(rn + 16);
            gather(r1.r + (int32_t)a.row_begin, j1a, j1b, k1a, k1b);
            load_w(r1, w1a, w1b);
        }
        // ---- fold vertex n ----
        const int32_t vk = rc.r + (int32_t)a.row_begin;
        const int32_t cs = warp_fold<W, SLOTS, O32>(a, tab, lane, lanes_below, r_o(rc), dk, vk, rc.ci, k0a, k0b, w0a, w0b, ep);
        if (accept_move(cs, rc.ci, pl)) {
            c_ch += 1;
            c_che += dk;
            if (lane == 0) a.lab_out[vk] = cs;
            if (!SYNC) {
                // vertex n+1's labels were gathered before this write: patch them
                if (j1a == vk) k1a = cs;
                if (j1b == vk) k1b = cs;
            }
            if (j0a >= 0) a.flag_out[j0a] = 1;            // mark neighbours unprocessed
            if (j0b >= 0) a.flag_out[j0b] = 1;
            for (uint32_t b = 64 + lane; b < dk; b += 32) a.flag_out[a.indices[at(r_o(rc), b)]] = 1;
        }
        // rotate the pipeline
        j0a = j1a; j0b = j1b; k0a = k1a; k0b = k1b; w0a = w1a; w0b = w1b;
        j1a = j2a; j1b = j2b;
      }
    }
done:
    if (lane == 0 && c_ch) {
        atomicAdd(&bctr[0], (unsigned long long)c_ch);
        atomicAdd(&bctr[1], (unsigned long long)c_che);
    }
    __syncthreads();
    if (threadIdx.x == 0 && bctr[0]) {
        atomicAdd(&a.ctr[0], bctr[0]);
        atomicAdd(&a.ctr[9 + bin], bctr[0]);
        atomicAdd(&a.ctr[13 + bin], bctr[1]);
    }
}

// ---------------------------------------------------------------------------
// block-per-vertex kernel: one CTA of 8 warps per vertex
// (degree wide_degree <= D < giant_degree), the vertex's table -- p1 =
// nextPow2(D)-1 slots as in PAPER.md:208 -- in shared memory.  The row is
// staged by TMA: one thread issues a 1-D bulk copy (cp.async.bulk, mbarrier
// completion) of the NEXT vertex's indices (and weights) into the other of
// two shared row buffers while the CTA folds this one, so no thread waits
// on a dependent CSR load; all label gathers C[j] of a row are issued
// before its fold (up to R per thread, in registers).  Per 32-entry batch a
// warp folds equal labels with match_any; the group leader claims the
// label's slot (Algorithm 2 probing, atomicCAS) and adds the group total --
// an integer count (exact for unit weights, native shared atomicAdd) or,
// for other weights, a float atomicAdd.  hashtableMaxKey is a scan of the
// table's p1 slots (ties: smallest label, R6).
// ---------------------------------------------------------------------------
constexpr int kBlkThreads = 256;

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}" ::"r"(bar), "r"(parity) : "memory");
}
// 1-D bulk copy global -> shared (TMA), completion counted on mbarrier `bar`
__device__ __forceinline__ void tma_load_1d(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}

// NT threads per CTA (one vertex); R: label gathers per thread (rows of up to R * NT entries);
// rowcap: entries per row buffer (>= max degree + 4, multiple of 4);
// cap: table slots (>= p1 of the largest degree).
template <bool SYNC, bool W, int R, int NT>
__global__ void __launch_bounds__(NT) k_block(SweepArgs a, const VRec *__restrict__ recs,
                                                        const unsigned long long *__restrict__ count, int cap,
                                                        int rowcap) {
    extern __shared__ __align__(16) uint8_t dyn_b[];
    int32_t *Hk = reinterpret_cast<int32_t *>(dyn_b);                 // keys (kEmpty = free)
    uint32_t *Hc = reinterpret_cast<uint32_t *>(Hk + cap);            // unit-weight counts
    float *Hf = reinterpret_cast<float *>(Hc + cap);                  // other weights
#if NULPA_BLOCK_LIST
    uint32_t *Hlist = reinterpret_cast<uint32_t *>(Hf + cap);         // slots claimed by this vertex
    int32_t *rowi = reinterpret_cast<int32_t *>(Hlist + cap);         // 2 index buffers of rowcap
    __shared__ uint32_t s_nlist;
#else
    int32_t *rowi = reinterpret_cast<int32_t *>(Hf + cap);            // 2 index buffers of rowcap
#endif
    float *roww = reinterpret_cast<float *>(rowi + 2 * rowcap);       // 2 weight buffers (W)
    __shared__ __align__(8) uint64_t s_bar[2];
    __shared__ uint64_t s_best[NT / 32];
    __shared__ int s_changed;
#if NULPA_MAJORITY
    __shared__ uint32_t s_maj[3];            // own-label count, neighbour count, non-unit weight seen
#endif
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(&s_bar[0]);
    const int64_t n = (int64_t)*count;
    unsigned long long n_changed = 0, n_changed_edges = 0;
    auto r_o = [](const VRec &r) -> int64_t { return (int64_t)(((uint64_t)(r.o_hi_deg & 0xFFFFu) << 32) | r.o_lo); };
    auto r_d = [](const VRec &r) -> uint32_t { return r.o_hi_deg >> 16; };
    // the row of record r into buffer b (one thread): indices [o & ~3, ...)
    auto stage = [&](const VRec &r, int b) {
        const int64_t o = r_o(r), o0 = o & ~INT64_C(3);
        const uint32_t ents = (uint32_t)(((o + r_d(r) - o0) + 3) & ~INT64_C(3));
        const uint32_t bar = bar0 + 8u * b;
        mbar_expect_tx(bar, ents * 4u * (W ? 2u : 1u));
        tma_load_1d((uint32_t)__cvta_generic_to_shared(rowi + b * rowcap), a.indices + o0, ents * 4u, bar);
        if (W) tma_load_1d((uint32_t)__cvta_generic_to_shared(roww + b * rowcap), a.weights + o0, ents * 4u, bar);
    };
    if (threadIdx.x == 0) {
        mbar_init(bar0, 1);
        mbar_init(bar0 + 8, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
#if NULPA_MAJORITY
    if (threadIdx.x < 3) s_maj[threadIdx.x] = 0;
#endif
#if NULPA_BLOCK_LIST
    // the table is cleared once; afterwards every vertex resets the slots it
    // claimed (listed in Hlist) while it scans them for hashtableMaxKey
    for (int q = threadIdx.x; q < cap; q += NT) {
        Hk[q] = kEmpty;
        Hc[q] = 0;
        Hf[q] = 0.0f;
    }
    if (threadIdx.x == 0) s_nlist = 0;
#endif
    __syncthreads();
    if (threadIdx.x == 0 && (int64_t)blockIdx.x < n) stage(recs[blockIdx.x], 0);
    int i = 0;
    for (int64_t k = blockIdx.x; k < n; k += gridDim.x, ++i) {
        const int b = i & 1;
        const VRec rc = recs[k];
        if (threadIdx.x == 0 && k + gridDim.x < n) {
            // buffer b^1 was last read by vertex i-1 (done: trailing __syncthreads)
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            stage(recs[k + gridDim.x], b ^ 1);
        }
        const uint32_t deg = r_d(rc);
        const int64_t v = rc.r + a.row_begin;
        Hash h;
        h.init(deg);
#if !NULPA_BLOCK_LIST
        for (uint32_t q = threadIdx.x; q < h.p1; q += NT) {   // hashtableClear
            Hk[q] = kEmpty;
            Hc[q] = 0;
            Hf[q] = 0.0f;
        }
#endif
        mbar_wait(bar0 + 8u * b, (uint32_t)(i >> 1) & 1u);
        const int32_t *ri = rowi + b * rowcap + (r_o(rc) & 3);
        const float *rw = roww + b * rowcap + (r_o(rc) & 3);
        // every label gather of the row in flight at once
        int32_t key[R];
        float w[R];
#pragma unroll
        for (int u = 0; u < R; ++u) {
            const uint32_t e = (uint32_t)(u * NT) + threadIdx.x;
            key[u] = kEmpty;
            w[u] = 1.0f;
            if (e < deg) {
                const int32_t j = ri[e];
                if (j != (int32_t)v) key[u] = a.lab_in[j];          // "if j = i continue"
                if (W) w[u] = rw[e];
            }
        }
#if NULPA_MAJORITY
        // strict majority of the vertex's own label (unit weights, past the
        // first sweep): it is hashtableMaxKey and the vertex does not move --
        // no table work (see warp_fold)
        if (!a.first) {
            uint32_t own = 0, tot = 0;
            bool unit = true;
#pragma unroll
            for (int u = 0; u < R; ++u) {
                if ((uint32_t)(u * NT) + (uint32_t)(wid * 32) >= deg) break;   // warp-uniform
                own += __popc(__ballot_sync(0xFFFFFFFFu, key[u] == rc.ci));
                tot += __popc(__ballot_sync(0xFFFFFFFFu, key[u] != kEmpty));
                if (W) unit = unit && __all_sync(0xFFFFFFFFu, key[u] == kEmpty || w[u] == 1.0f);
            }
            if (lane == 0 && tot) {
                atomicAdd(&s_maj[0], own);
                atomicAdd(&s_maj[1], tot);
                if (!unit) s_maj[2] = 1;
            }
        }
#endif
        __syncthreads();                                             // table cleared
#if NULPA_MAJORITY
        const bool maj = !a.first && s_maj[2] == 0 && 2 * s_maj[0] > s_maj[1];
#else
        constexpr bool maj = false;
#endif
#pragma unroll
        for (int u = 0; u < R; ++u) {
            if (maj) break;
            if ((uint32_t)(u * NT) + (uint32_t)(wid * 32) >= deg) break;   // warp-uniform
            const unsigned grp = __match_any_sync(0xFFFFFFFFu, key[u]);
            const bool leader = key[u] != kEmpty && (grp & ((1u << lane) - 1)) == 0;
            const bool eq = !W || __all_sync(0xFFFFFFFFu, key[u] == kEmpty || w[u] == 1.0f);
            float x = 0.0f;
            if (!eq) {
                const unsigned maxn = __reduce_max_sync(0xFFFFFFFFu, key[u] != kEmpty ? (unsigned)__popc(grp) : 1u);
                x = maxn > 1 ? group_sum(grp, w[u], maxn) : w[u];
            }
            uint32_t slot = 0;
            bool fresh = false;
            if (leader) {
                slot = ht_claim(Hk, h, key[u], &fresh);
                if (eq) atomicAdd(&Hc[slot], (uint32_t)__popc(grp));
                else atomicAdd(&Hf[slot], x);
            }
#if NULPA_BLOCK_LIST
            // list the newly claimed slots: one shared atomic per warp and batch
            const unsigned fm = __ballot_sync(0xFFFFFFFFu, fresh);
            if (fm) {
                uint32_t base = 0;
                if (lane == __ffs(fm) - 1) base = atomicAdd(&s_nlist, (uint32_t)__popc(fm));
                base = __shfl_sync(0xFFFFFFFFu, base, __ffs(fm) - 1);
                if (fresh) Hlist[base + __popc(fm & ((1u << lane) - 1))] = slot;
            }
#endif
        }
        __syncthreads();                                             // table complete
        // hashtableMaxKey: (total, smallest label) as one 64-bit max
        uint64_t best = 0;
#if NULPA_BLOCK_LIST
        const uint32_t nl = s_nlist;
        for (uint32_t q = threadIdx.x; q < nl; q += NT) {
            const uint32_t sl = Hlist[q];
            const int32_t kk = Hk[sl];
            const float t = __fadd_rn((float)Hc[sl], Hf[sl]);
            const uint64_t c = ((uint64_t)(__float_as_uint(t) + 1) << 32) | (uint32_t)~kk;
            best = c > best ? c : best;
            Hk[sl] = kEmpty;                                         // hashtableClear of the claimed slots
            Hc[sl] = 0;
            Hf[sl] = 0.0f;
        }
#else
        for (uint32_t q = threadIdx.x; q < h.p1; q += NT) {
            const int32_t kk = Hk[q];
            if (kk == kEmpty) continue;
            const float t = __fadd_rn((float)Hc[q], Hf[q]);
            const uint64_t c = ((uint64_t)(__float_as_uint(t) + 1) << 32) | (uint32_t)~kk;
            best = c > best ? c : best;
        }
#endif
        best = warp_max_u64(best);
        if (lane == 0) s_best[wid] = best;
        __syncthreads();
        if (threadIdx.x == 0) {
            uint64_t bb = 0;
            for (int q = 0; q < NT / 32; ++q) bb = s_best[q] > bb ? s_best[q] : bb;
            const int32_t cs = maj ? rc.ci : bb ? (int32_t)~(uint32_t)bb : kEmpty;
            const int ch = accept_move(cs, rc.ci, sweep_pl(a));
            if (ch) a.lab_out[v] = cs;
            s_changed = ch;
#if NULPA_BLOCK_LIST
            s_nlist = 0;                                             // the next vertex's claims come after two more barriers
#endif
#if NULPA_MAJORITY
            s_maj[0] = s_maj[1] = s_maj[2] = 0;                      // likewise the next vertex's counts
#endif
            n_changed += ch;
            n_changed_edges += ch ? deg : 0;
        }
        __syncthreads();
        if (s_changed)
            for (uint32_t e = threadIdx.x; e < deg; e += NT) a.flag_out[ri[e]] = 1;
        __syncthreads();                                             // row buffer b and s_changed reusable
    }
    if (threadIdx.x == 0 && n_changed) {
        atomicAdd(&a.ctr[0], n_changed);
        atomicAdd(&a.ctr[9 + 2], n_changed);
        atomicAdd(&a.ctr[13 + 2], n_changed_edges);
    }
}

// ---------------------------------------------------------------------------
// giant vertices (degree >= giant_degree): the row is cut into chunks of
// kGiantChunk edges, one CTA per chunk.  Each CTA pre-aggregates its chunk in
// a shared-memory table (recording the slots it claims), then folds the
// distinct (label, weight) pairs into the vertex's GLOBAL-memory table
// (p1 = nextPow2(D)-1 slots) with atomicAdd.  Weights are
// non-negative (R12), so a label's running totals only grow and the largest
// total any fold returns is hashtableMaxKey: each CTA folds the best
// (total, tie rank) it saw into best[gi] with one 64-bit atomicMax -- no
// scan of the global table.  Newly claimed global slots go to an occupied
// list, which k_giant_finish clears (and, for moved vertices, the chunk's
// neighbours are marked there too).
// ---------------------------------------------------------------------------
struct GiantArgs {
    const int32_t *verts;        // [ng] local row ids
    const int32_t *chunk_g;      // [nc] giant index of the chunk
    const int64_t *chunk_e0;     // [nc] first edge of the chunk
    const int64_t *chunk_e1;     // [nc] end edge of the chunk
    const int64_t *table_off;    // [ng] first slot of the vertex's global table
    int32_t *keys;               // global tables
    float *vals;
    int32_t *occ;                // occupied-slot lists (same offsets)
    int32_t *occ_n;              // [ng]
    uint8_t *active;             // [ng]
    uint8_t *changed;            // [ng]
    unsigned long long *best;    // [ng] packed (weight, tie rank) maximum
    unsigned long long *maj;     // [3 ng] own-label count, neighbour count, non-unit weights seen (majority shortcut)
};

template <bool SYNC>
__global__ void k_giant_snapshot(SweepArgs a, GiantArgs g, int64_t ng) {
    int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= ng) return;
    int64_t v = g.verts[k] + a.row_begin;
    uint8_t f = a.flag_in[v];
    g.active[k] = f ? 1 : 0;
    g.changed[k] = 0;
    g.best[k] = 0;
    g.occ_n[k] = 0;
    g.maj[3 * k] = g.maj[3 * k + 1] = g.maj[3 * k + 2] = 0;
    if (!SYNC && f) a.flag_in[v] = 0;
}

#if NULPA_MAJORITY
// Majority shortcut for giant vertices (every sweep but the first after a
// reset): one pass over the active giants' rows counting the neighbours that
// hold the vertex's own label, the neighbours, and non-unit weights; a giant
// whose own label holds a strict majority (unit weights) skips the table
// fold and keeps its label (k_giant_accumulate / k_giant_decide).
template <bool W>
__global__ void __launch_bounds__(kBlockThreads) k_giant_count(SweepArgs a, GiantArgs g) {
    const int64_t c = blockIdx.x;
    const int32_t gi = g.chunk_g[c];
    if (!g.active[gi]) return;
    const int64_t v = g.verts[gi] + a.row_begin;
    const int32_t ci = a.lab_in[v];
    const int64_t e0 = g.chunk_e0[c], e1 = g.chunk_e1[c];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    uint32_t own = 0, tot = 0, nonunit = 0;
    for (int64_t b = e0 + wid * 32; b < e1; b += 2 * kBlockThreads) {
        int32_t j[2] = {-1, -1};
        float w[2] = {1.0f, 1.0f};
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            const int64_t e = b + u * kBlockThreads + lane;
            if (e < e1) {
                j[u] = ld_stream(a.indices + e);
                if (W) w[u] = ld_stream(a.weights + e);
            }
        }
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            const int32_t key = (j[u] >= 0 && j[u] != (int32_t)v) ? a.lab_in[j[u]] : kEmpty;
            own += __popc(__ballot_sync(0xFFFFFFFFu, key == ci));
            tot += __popc(__ballot_sync(0xFFFFFFFFu, key != kEmpty));
            if (W) nonunit += __popc(__ballot_sync(0xFFFFFFFFu, key != kEmpty && w[u] != 1.0f));
        }
    }
    if (lane == 0 && tot) {
        atomicAdd(&g.maj[3 * gi], (unsigned long long)own);
        atomicAdd(&g.maj[3 * gi + 1], (unsigned long long)tot);
        if (nonunit) atomicAdd(&g.maj[3 * gi + 2], (unsigned long long)nonunit);
    }
}
#endif
__device__ __forceinline__ bool giant_majority(const SweepArgs &a, const GiantArgs &g, int64_t gi) {
#if NULPA_MAJORITY
    return !a.first && g.maj[3 * gi + 2] == 0 && 2 * g.maj[3 * gi] > g.maj[3 * gi + 1];
#else
    return false;
#endif
}

template <bool SYNC, bool W>
__global__ void __launch_bounds__(kBlockThreads) k_giant_accumulate(SweepArgs a, GiantArgs g) {
    extern __shared__ int32_t dyn[];
    int32_t *Hk = dyn;
    float *Hv = reinterpret_cast<float *>(dyn + kGiantCap);
    uint16_t *s_occ = reinterpret_cast<uint16_t *>(dyn + 2 * kGiantCap);   // claimed slots (<= kGiantChunk)
    __shared__ int s_nocc;
    __shared__ uint64_t red[kBlockThreads / 32];
    const int64_t c = blockIdx.x;
    const int32_t gi = g.chunk_g[c];
    if (!g.active[gi]) return;
    const int32_t r = g.verts[gi];
    const int64_t v = r + a.row_begin;
    const int64_t e0 = g.chunk_e0[c], e1 = g.chunk_e1[c];
    if (giant_majority(a, g, gi)) {                        // no table fold (k_giant_count)
        if (threadIdx.x == 0) atomicAdd(&a.ctr[5 + 3], (unsigned long long)(e1 - e0));
        return;
    }
    for (int s = threadIdx.x; s < kGiantCap; s += kBlockThreads) {
        Hk[s] = kEmpty;
        Hv[s] = 0.0f;
    }
    if (threadIdx.x == 0) s_nocc = 0;
    __syncthreads();
    Hash hc;
    hc.init((uint32_t)(e1 - e0));
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    // two 32-edge batches per warp per step: both index loads, then both gathers in flight
    for (int64_t b = e0 + wid * 32; b < e1; b += 2 * kBlockThreads) {
        int32_t key[2] = {kEmpty, kEmpty};
        float w[2] = {0.0f, 0.0f};
        int32_t j[2] = {-1, -1};
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            const int64_t e = b + u * kBlockThreads + lane;
            if (e < e1) {
                j[u] = ld_stream(a.indices + e);
                if (W) w[u] = ld_stream(a.weights + e);
            }
        }
#pragma unroll
        for (int u = 0; u < 2; ++u)
            if (j[u] >= 0 && j[u] != (int32_t)v) key[u] = a.lab_in[j[u]];
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            if (b + u * kBlockThreads >= e1) break;
            const unsigned grp = __match_any_sync(0xFFFFFFFFu, key[u]);
            const bool leader = key[u] != kEmpty && lane == __ffs(grp) - 1;
            float sum;
            if (W) {
                const unsigned valid = __ballot_sync(0xFFFFFFFFu, key[u] != kEmpty);
                const float wr = __shfl_sync(0xFFFFFFFFu, w[u], valid ? __ffs(valid) - 1 : 0);
                if (__all_sync(0xFFFFFFFFu, key[u] == kEmpty || w[u] == wr)) {
                    sum = (float)__popc(grp) * w[u];
                } else {
                    const unsigned maxn = __reduce_max_sync(0xFFFFFFFFu, key[u] != kEmpty ? (unsigned)__popc(grp) : 1u);
                    sum = maxn > 1 ? group_sum(grp, w[u], maxn) : w[u];
                }
            } else {
                sum = (float)__popc(grp);
            }
            if (leader) {
                uint32_t slot;
                if (ht_accumulate(Hk, Hv, hc, key[u], sum, &slot)) s_occ[atomicAdd(&s_nocc, 1)] = (uint16_t)slot;
            }
        }
    }
    __syncthreads();
    Hash hg;
    hg.init((uint32_t)(a.offsets[r + 1] - a.offsets[r]));
    TieOrder to;
    to.init(hg);
    int32_t *gk = g.keys + g.table_off[gi];
    float *gv = g.vals + g.table_off[gi];
    int32_t *occ = g.occ + g.table_off[gi];
    uint64_t best = 0;
    const int nocc = s_nocc;
    for (int q = threadIdx.x; q < nocc; q += kBlockThreads) {
        const uint32_t s = s_occ[q];
        const int32_t k = Hk[s];
        uint32_t slot;
        float total;
        if (ht_accumulate(gk, gv, hg, k, Hv[s], &slot, &total)) occ[atomicAdd(&g.occ_n[gi], 1)] = (int32_t)slot;
        const uint64_t cd = pack_cand(total, k, to);
        best = cd > best ? cd : best;
    }
    best = warp_max_u64(best);
    if (lane == 0) red[wid] = best;
    __syncthreads();
    if (wid == 0) {
        uint64_t bb = lane < kBlockThreads / 32 ? red[lane] : 0;
        bb = warp_max_u64(bb);
        if (lane == 0 && bb) atomicMax(&g.best[gi], (unsigned long long)bb);
    }
    if (threadIdx.x == 0) atomicAdd(&a.ctr[5 + 3], (unsigned long long)(e1 - e0));
}

// the move rule for every giant vertex (one thread each)
template <bool SYNC>
__global__ void k_giant_decide(SweepArgs a, GiantArgs g, int64_t ng) {
    const int64_t gi = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (gi >= ng || !g.active[gi]) return;
    const int32_t r = g.verts[gi];
    const int64_t v = r + a.row_begin;
    const int64_t deg = a.offsets[r + 1] - a.offsets[r];
    Hash h;
    h.init((uint32_t)deg);
    TieOrder to;
    to.init(h);
    const unsigned long long b = g.best[gi];
    const int32_t cs = giant_majority(a, g, gi) ? a.lab_in[v] : b ? cand_label(b, to) : kEmpty;
    const bool ch = accept_move(cs, a.lab_in[v], sweep_pl(a));
    if (ch) {
        a.lab_out[v] = cs;
        g.changed[gi] = 1;
        atomicAdd(&a.ctr[0], 1ull);
        atomicAdd(&a.ctr[9 + 3], 1ull);
        atomicAdd(&a.ctr[13 + 3], (unsigned long long)deg);
    }
    atomicAdd(&a.ctr[1 + 3], 1ull);
}

// per chunk CTA: clear its slice of the vertex's occupied list (hashtableClear
// of the used slots) and, if the vertex moved, mark the chunk's neighbours
__global__ void __launch_bounds__(kBlockThreads) k_giant_finish(SweepArgs a, GiantArgs g) {
    const int64_t c = blockIdx.x;
    const int32_t gi = g.chunk_g[c];
    if (!g.active[gi]) return;
    const int32_t r = g.verts[gi];
    const int64_t kc = (g.chunk_e0[c] - a.offsets[r]) / kGiantChunk;
    int32_t *gk = g.keys + g.table_off[gi];
    float *gv = g.vals + g.table_off[gi];
    const int32_t *occ = g.occ + g.table_off[gi];
    const int64_t cnt = g.occ_n[gi];
    const int64_t q0 = kc * kGiantChunk, q1 = q0 + kGiantChunk < cnt ? q0 + kGiantChunk : cnt;
    for (int64_t q = q0 + threadIdx.x; q < q1; q += kBlockThreads) {
        const int32_t sl = occ[q];
        gk[sl] = kEmpty;
        gv[sl] = 0.0f;
    }
    if (g.changed[gi])
        for (int64_t e = g.chunk_e0[c] + threadIdx.x; e < g.chunk_e1[c]; e += kBlockThreads)
            a.flag_out[a.indices[e]] = 1;
}

// ---------------------------------------------------------------------------
// state / binning kernels
// ---------------------------------------------------------------------------
__global__ void k_init_state(int32_t *labels, uint8_t *flags, int64_t n) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        labels[i] = (int32_t)i;     // C <- [0 .. |V|)
        flags[i] = 1;               // all vertices unprocessed
    }
}

constexpr int kBinTile = 256;       // rows per tile (one per thread)
constexpr int kBinTiles = 4;        // tiles per CTA

__device__ __forceinline__ int bin_of(int64_t d, int32_t t1, int32_t t2, int32_t t3) {
    return d == 0 ? -1 : d < t1 ? 0 : d < t2 ? 1 : d < t3 ? 2 : 3;
}

__global__ void __launch_bounds__(kBinTile) k_bin_count(const int64_t *offsets, int64_t n, int32_t t1, int32_t t2,
                                                        int32_t t3, int64_t *counts, unsigned long long *edges,
                                                        unsigned long long *maxdeg) {
    __shared__ int64_t c[4];
    __shared__ unsigned long long ed[4], md[4];
    if (threadIdx.x < 4) {
        c[threadIdx.x] = 0;
        ed[threadIdx.x] = 0;
        md[threadIdx.x] = 0;
    }
    __syncthreads();
    for (int k = 0; k < kBinTiles; ++k) {
        int64_t r = ((int64_t)blockIdx.x * kBinTiles + k) * kBinTile + threadIdx.x;
        if (r < n) {
            int64_t d = offsets[r + 1] - offsets[r];
            int b = bin_of(d, t1, t2, t3);
            if (b >= 0) {
                atomicAdd((unsigned long long *)&c[b], 1ull);
                atomicAdd(&ed[b], (unsigned long long)d);
                atomicMax(&md[b], (unsigned long long)d);
            }
        }
    }
    __syncthreads();
    if (threadIdx.x < 4) {
        counts[(int64_t)blockIdx.x * 4 + threadIdx.x] = c[threadIdx.x];
        atomicAdd(&edges[threadIdx.x], ed[threadIdx.x]);
        atomicMax(&maxdeg[threadIdx.x], md[threadIdx.x]);
    }
}

// exclusive scan of counts[nb][4] per bin (single CTA of 1024 threads)
__global__ void __launch_bounds__(1024) k_bin_scan(int64_t *counts, int64_t nb, int64_t *totals) {
    __shared__ int64_t ws[32];
    __shared__ int64_t carry_s;
    for (int b = 0; b < 4; ++b) {
        if (threadIdx.x == 0) carry_s = 0;
        __syncthreads();
        for (int64_t base = 0; base < nb; base += 1024) {
            int64_t i = base + threadIdx.x;
            int64_t x = i < nb ? counts[i * 4 + b] : 0;
            // inclusive warp scan
            int64_t y = x;
            for (int o = 1; o < 32; o <<= 1) {
                int64_t z = __shfl_up_sync(0xFFFFFFFFu, y, o);
                if ((threadIdx.x & 31) >= o) y += z;
            }
            if ((threadIdx.x & 31) == 31) ws[threadIdx.x >> 5] = y;
            __syncthreads();
            if (threadIdx.x < 32) {
                int64_t s = ws[threadIdx.x];
                for (int o = 1; o < 32; o <<= 1) {
                    int64_t z = __shfl_up_sync(0xFFFFFFFFu, s, o);
                    if (threadIdx.x >= o) s += z;
                }
                ws[threadIdx.x] = s;
            }
            __syncthreads();
            int64_t warp_prefix = (threadIdx.x >> 5) ? ws[(threadIdx.x >> 5) - 1] : 0;
            int64_t carry = carry_s;
            if (i < nb) counts[i * 4 + b] = carry + warp_prefix + y - x;
            __syncthreads();
            if (threadIdx.x == 1023) carry_s = carry + warp_prefix + y;
            __syncthreads();
        }
        if (threadIdx.x == 0) totals[b] = carry_s;
        __syncthreads();
    }
}

struct BinLists {
    int32_t *l[4];
};

__global__ void __launch_bounds__(kBinTile) k_bin_scatter(const int64_t *offsets, int64_t n, int32_t t1, int32_t t2,
                                                          int32_t t3, const int64_t *base, BinLists lists) {
    __shared__ int32_t wc[kBinTile / 32][4];
    __shared__ int64_t run[4];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    if (threadIdx.x < 4) run[threadIdx.x] = base[(int64_t)blockIdx.x * 4 + threadIdx.x];
    __syncthreads();
    for (int k = 0; k < kBinTiles; ++k) {
        int64_t r = ((int64_t)blockIdx.x * kBinTiles + k) * kBinTile + threadIdx.x;
        int b = -1;
        if (r < n) b = bin_of(offsets[r + 1] - offsets[r], t1, t2, t3);
        unsigned lt = (1u << lane) - 1;
        int my_rank = 0;
        for (int q = 0; q < 4; ++q) {
            unsigned m = __ballot_sync(0xFFFFFFFFu, b == q);
            if (b == q) my_rank = __popc(m & lt);
            if (lane == 0) wc[wid][q] = __popc(m);
        }
        __syncthreads();
        if (b >= 0) {
            int64_t off = run[b];
            for (int w = 0; w < wid; ++w) off += wc[w][b];
            lists.l[b][off + my_rank] = (int32_t)r;
        }
        __syncthreads();
        if (threadIdx.x < 4) {
            int64_t s = 0;
            for (int w = 0; w < kBinTile / 32; ++w) s += wc[w][threadIdx.x];
            run[threadIdx.x] += s;
        }
        __syncthreads();
    }
}

// ID locality of the graph (first-sweep schedule, DESIGN.md "Quality
// notes"): over `ns` sampled rows (every `step`-th), acc[0] += CSR entries,
// acc[1] += entries whose neighbour ID is within kNear of the row's ID.
constexpr int64_t kNear = 2048;
__global__ void k_locality(const int64_t *__restrict__ offsets, const int32_t *__restrict__ indices, int64_t row_begin,
                           int64_t step, int64_t ns, unsigned long long *acc) {
    unsigned long long tot = 0, near = 0;
    for (int64_t s = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; s < ns; s += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = s * step, v = r + row_begin;
        const int64_t e1 = min(offsets[r + 1], offsets[r] + 64);    // up to 64 entries per sampled row
        for (int64_t e = offsets[r]; e < e1; ++e) {
            const int64_t d = (int64_t)indices[e] - v;
            near += d >= -kNear && d <= kNear;
            ++tot;
        }
    }
    atomicAdd(&acc[0], tot);
    atomicAdd(&acc[1], near);
}

__global__ void k_gather_degrees(const int64_t *offsets, const int32_t *rows, int64_t n, int64_t *out) {
    int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k < n) {
        out[k] = offsets[rows[k] + 1] - offsets[rows[k]];
        out[n + k] = offsets[rows[k]];
    }
}

// ---------------------------------------------------------------------------
// modularity (Eq. 1, second form, R11), float64
// ---------------------------------------------------------------------------
// K_i = sum_j w_ij for every row (float64), computed once per handle; acc[1] += 2m
template <bool W>
__global__ void __launch_bounds__(256) k_mod_degrees(const int64_t *__restrict__ offsets, const float *__restrict__ weights,
                                                     int64_t n_rows, double *K, double *acc) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x / 32);
    double tot = 0.0;
    for (int64_t r = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); r < n_rows; r += nw) {
        double k = 0.0;
        if (W) {
            for (int64_t e = offsets[r] + lane; e < offsets[r + 1]; e += 32) k += (double)weights[e];
#pragma unroll
            for (int o = 16; o; o >>= 1) k += __shfl_xor_sync(0xFFFFFFFFu, k, o);
        } else {
            k = (double)(offsets[r + 1] - offsets[r]);
        }
        if (lane == 0) {
            K[r] = k;
            tot += k;
        }
    }
    if (lane == 0) atomicAdd(&acc[1], tot);
}

// acc[0] += sigma_intra = sum over CSR entries (i,j) with C_i = C_j of w_ij.
// A warp takes 32 consecutive rows and streams their CSR entries as one flat,
// coalesced range (32 entries per lane step, two steps in flight); an
// entry's row is found by a 5-step binary search over the 33 row offsets
// held one per lane (shuffles), its label compared with the gathered C_j.
// Per-lane float64 partial sums, reduced once at the end.
template <bool W>
__global__ void __launch_bounds__(256) k_mod_intra(const int64_t *__restrict__ offsets, const int32_t *__restrict__ indices,
                                                   const float *__restrict__ weights, const int32_t *__restrict__ labels,
                                                   int64_t n_rows, int64_t row_begin, double *acc) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = (int64_t)gridDim.x * (blockDim.x / 32);
    const int64_t nchunks = (n_rows + 31) / 32;
    double in = 0.0;
    for (int64_t c = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); c < nchunks; c += nw) {
        const int64_t r0 = c * 32, r = r0 + lane;
        const int64_t o_abs = offsets[min(r, n_rows)];
        const int32_t cl = r < n_rows ? labels[r + row_begin] : 0;
        const int64_t e0 = __shfl_sync(0xFFFFFFFFu, o_abs, 0);
        const uint32_t ol = (uint32_t)(o_abs - e0);                   // row starts relative to the chunk
        const uint32_t len = (uint32_t)(offsets[min(r0 + 32, n_rows)] - e0);
        const int32_t nr = n_rows - r0 < 32 ? (int32_t)(n_rows - r0) : 32;
        auto row_of = [&](uint32_t e) -> int32_t {                   // largest k < nr with start(k) <= e
            int32_t k = 0;
#pragma unroll
            for (int st = 16; st; st >>= 1) {
                const int32_t t = k + st;
                const uint32_t ot = __shfl_sync(0xFFFFFFFFu, ol, t & 31);
                if (t < nr && ot <= e) k = t;
            }
            return k;
        };
        constexpr int UM = 4;                                         // entries per lane in flight
        for (uint32_t base = 0; base < len; base += 32 * UM) {
            int32_t j[UM], lb[UM];
            float w[UM];
            bool v[UM];
#pragma unroll
            for (int u = 0; u < UM; ++u) {
                const uint32_t e = base + 32 * u + lane;
                v[u] = e < len;
                j[u] = v[u] ? ld_stream(indices + e0 + e) : 0;
                w[u] = W && v[u] ? ld_stream(weights + e0 + e) : 1.0f;
            }
#pragma unroll
            for (int u = 0; u < UM; ++u) lb[u] = v[u] ? labels[j[u]] : 0;
#pragma unroll
            for (int u = 0; u < UM; ++u) {
                const int32_t cr = __shfl_sync(0xFFFFFFFFu, cl, row_of(base + 32 * u + lane));
                if (v[u] && lb[u] == cr) in += W ? (double)w[u] : 1.0;
            }
        }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) in += __shfl_xor_sync(0xFFFFFFFFu, in, o);
    __shared__ double s_in[8];
    if (lane == 0) s_in[threadIdx.x >> 5] = in;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0;
        for (int w = 0; w < (int)(blockDim.x / 32); ++w) t += s_in[w];
        atomicAdd(&acc[0], t);
    }
}

// Sigma[C_i] += K_i, one thread per row; rows of a warp holding the same
// label are summed first (match_any + pairwise tree) so a community costs
// one atomicAdd per warp instead of one per vertex.
__device__ __forceinline__ double group_sum_d(unsigned grp, double x, unsigned maxn) {
    const int lane = threadIdx.x & 31;
    const unsigned rank = __popc(grp & ((1u << lane) - 1));
    const unsigned above = lane == 31 ? 0u : grp & (0xFFFFFFFEu << lane);
    int nxt = above ? __ffs(above) - 1 : 32;
    for (unsigned d = 1; d < maxn; d <<= 1) {
        const double y = __shfl_sync(0xFFFFFFFFu, x, nxt & 31);
        const int n2 = __shfl_sync(0xFFFFFFFFu, nxt, nxt & 31);
        if ((rank & (2 * d - 1)) == 0 && nxt < 32) x += y;
        nxt = nxt < 32 ? n2 : 32;
    }
    return x;
}
__global__ void __launch_bounds__(256) k_mod_sigma(const double *__restrict__ K, const int32_t *__restrict__ labels,
                                                   int64_t n_rows, int64_t row_begin, double *Sigma) {
    const int lane = threadIdx.x & 31;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n_rows; base += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = base + threadIdx.x;
        const int32_t c = r < n_rows ? labels[r + row_begin] : -1;
        const double k = r < n_rows ? K[r] : 0.0;
        const unsigned grp = __match_any_sync(0xFFFFFFFFu, c);
        const unsigned maxn = __reduce_max_sync(0xFFFFFFFFu, (unsigned)__popc(grp));
        const double s = maxn > 1 ? group_sum_d(grp, k, maxn) : k;
        if (c >= 0 && lane == __ffs(grp) - 1 && s != 0.0) atomicAdd(&Sigma[c], s);
    }
}

// acc[2] += sum_c Sigma_c^2 ; Sigma reset to 0 when `clear`
__global__ void __launch_bounds__(256) k_mod_finish(double *Sigma, int64_t n, double *acc, int clear) {
    double s = 0.0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        double x = Sigma[i];
        s += x * x;
        if (clear) Sigma[i] = 0.0;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xFFFFFFFFu, s, o);
    __shared__ double ws[8];
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
    __syncthreads();
    if (threadIdx.x == 0) {
        double t = 0;
        for (int w = 0; w < (int)(blockDim.x / 32); ++w) t += ws[w];
        atomicAdd(&acc[2], t);
    }
}

// SM count of the current device (cached per device ordinal)
int num_sms() {
    static int sms[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (!sms[dev]) {
        int n = 0;
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        sms[dev] = n > 0 ? n : 148;
    }
    return sms[dev];
}

// Input validation kernels (R12 and the label range of the C ABI).
// bad[0] += number of weights that are negative, NaN or infinite.
__global__ void k_check_weights(const float *__restrict__ w, int64_t m, unsigned long long *bad) {
    unsigned long long c = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < m; i += (int64_t)gridDim.x * blockDim.x) {
        const float x = w[i];
        c += !(x >= 0.0f && x <= 3.402823466e38f);      // false for NaN, < 0, +inf
    }
    c = __reduce_add_sync(0xFFFFFFFFu, (unsigned)c);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(bad, c);
}
// bad[0] += number of labels outside [0, n)
__global__ void k_check_labels(const int32_t *__restrict__ lab, int64_t n, unsigned long long *bad) {
    unsigned c = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        c += (lab[i] < 0 || (int64_t)lab[i] >= n);
    c = __reduce_add_sync(0xFFFFFFFFu, c);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(bad, (unsigned long long)c);
}

}  // namespace

// ---------------------------------------------------------------------------
// handle
// ---------------------------------------------------------------------------
struct nulpa_graph {
    int64_t n_rows = 0, n_global = 0, row_begin = 0, M = 0;
    int64_t *offsets = nullptr;
    int32_t *indices = nullptr;
    float *weights = nullptr;
    bool own_csr = false;
    int32_t *labels = nullptr;      // current labels (own or bound)
    uint8_t *flags = nullptr;       // current flags (own or bound)
    int32_t *own_labels = nullptr;
    uint8_t *own_flags = nullptr;
    int32_t *labels_prev = nullptr; // sync-mode snapshot
    uint8_t *flags_prev = nullptr;
    cudaStream_t stream = nullptr;
    // bins
    int32_t t1 = 0, t2 = 0, t3 = 0;
    bool bins_built = false;
    int32_t *bin_list[4] = {nullptr, nullptr, nullptr, nullptr};
    void *wrecs = nullptr;          // warp-bin frontier records (VRec [bin_n[1]])
    int32_t *trows = nullptr;       // thread-bin compacted frontier (rows [bin_n[0]]), k_tscan / k_tact
    unsigned long long *wranges = nullptr;   // SCHED_STEAL: one {next, end} group range per k_warp warp
    double locality = 0.0;          // share of sampled CSR entries j with |j - i| <= kNear (k_locality)
    void *brecs = nullptr;          // block-bin frontier records (VRec [2 * bin_n[2]]: warp part | CTA part)
    int64_t bin_n[4] = {0, 0, 0, 0};
    int64_t bin_e[4] = {0, 0, 0, 0};
    int64_t bin_maxdeg[4] = {0, 0, 0, 0};
    // giant
    int64_t n_chunks = 0;
    int32_t *chunk_g = nullptr;
    int64_t *chunk_e0 = nullptr, *chunk_e1 = nullptr, *table_off = nullptr;
    int32_t *gkeys = nullptr, *occ = nullptr, *occ_n = nullptr;
    float *gvals = nullptr;
    uint8_t *gactive = nullptr, *gchanged = nullptr;
    unsigned long long *gbest = nullptr;
    unsigned long long *gmaj = nullptr;      // [3 ng] majority-shortcut counts of the giant bin
    // counters
    unsigned long long *ctr = nullptr;       // device [kMaxIter+1][kCtr]
    unsigned long long *ctr_host = nullptr;  // pinned
    int sweep_slot = 0;                      // counter slot used by nulpa_sweep
    int64_t sweeps_since_reset = 0;          // selects first_sweep_block vs sweep_block
    // modularity scratch
    double *Sigma = nullptr;
    double *macc = nullptr;
    double *Kdeg = nullptr;                  // K_i (float64), cached by the first modularity call
    double two_m_local = 0.0;
    // timing
    cudaEvent_t ev[2 * 4 * (kMaxIter + 1)];
    cudaEvent_t ev_run[2];
    bool events = false;
    cudaStream_t side = nullptr;             // bin_order 2: block + giant bins
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    // device loop (nulpa_run without timing): [sweep 1.. + stop test] as a
    // CUDA graph with a conditional while node, built once per parameter set
    int32_t *loopvars = nullptr;             // device [4], see k_loop_step
    cudaGraph_t loop_graph = nullptr;
    cudaGraphExec_t loop_exec = nullptr;
    nulpa_params loop_p;                     // parameters the graph was captured with
    int loop_launches[4] = {0, 0, 0, 0};     // kernel launches of one loop body, per bin
    int loop_other = 0;
    int64_t runs = 0;                        // nulpa_run calls on this handle (the first uses the host loop)
    cudaStream_t cap = nullptr;              // capture stream of the device loop (the caller's may be the legacy stream)
    cudaStream_t hi = nullptr;               // bin_order 3: high-priority stream for the warp bin
    cudaEvent_t ev_mid = nullptr, ev_join2 = nullptr;
    nulpa_stats stats;
};

namespace {

// Device memory of every handle comes from one stream-ordered memory pool per
// device that keeps up to kPoolKeep bytes after they are freed: creating and
// destroying handles of the same size (the end-to-end path creates one per
// call) then reuses mapped memory instead of paying cudaMalloc / cudaFree of
// ~18 GB each time (measured 13-400 ms per call, varying).  Allocations are
// made on the legacy stream and synchronised before use on any stream; frees
// happen only after the handle's stream is idle.
constexpr uint64_t kPoolKeep = UINT64_C(48) << 30;
cudaMemPool_t device_pool() {
    static cudaMemPool_t pools[64] = {};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) return nullptr;
    if (!pools[dev]) {
        cudaMemPoolProps props = {};
        props.allocType = cudaMemAllocationTypePinned;
        props.location.type = cudaMemLocationTypeDevice;
        props.location.id = dev;
        if (cudaMemPoolCreate(&pools[dev], &props) != cudaSuccess) {
            pools[dev] = nullptr;
            return nullptr;
        }
        uint64_t keep = kPoolKeep;
        cudaMemPoolSetAttribute(pools[dev], cudaMemPoolAttrReleaseThreshold, &keep);
    }
    return pools[dev];
}

template <typename T>
int dalloc(T **p, size_t n) {
    if (n == 0) n = 1;
    cudaMemPool_t pool = device_pool();
    cudaError_t e = pool ? cudaMallocFromPoolAsync((void **)p, n * sizeof(T), pool, 0) : cudaMalloc((void **)p, n * sizeof(T));
    if (e == cudaSuccess && pool) e = cudaStreamSynchronize(0);
    if (e != cudaSuccess) {
        *p = nullptr;
        return fail(NULPA_ENOMEM, "device allocation of %zu bytes failed: %s", n * sizeof(T), cudaGetErrorString(e));
    }
    return NULPA_OK;
}

// callers make sure no kernel still uses p (handle stream synchronised)
void dfree(void *p) {
    if (p) cudaFreeAsync(p, 0);
}

void free_loop(nulpa_graph *g) {
    if (g->loop_exec) cudaGraphExecDestroy(g->loop_exec);
    if (g->loop_graph) cudaGraphDestroy(g->loop_graph);
    g->loop_exec = nullptr;
    g->loop_graph = nullptr;
}

void free_bins(nulpa_graph *g) {
    if (g->stream) cudaStreamSynchronize(g->stream);
    free_loop(g);
    dfree(g->wrecs);
    g->wrecs = nullptr;
    dfree(g->trows);
    g->trows = nullptr;
    dfree(g->wranges);
    g->wranges = nullptr;
    dfree(g->brecs);
    g->brecs = nullptr;
    for (int b = 0; b < 4; ++b) {
        dfree(g->bin_list[b]);
        g->bin_list[b] = nullptr;
        g->bin_n[b] = g->bin_e[b] = 0;
    }
    dfree(g->chunk_g);
    dfree(g->chunk_e0);
    dfree(g->chunk_e1);
    dfree(g->table_off);
    dfree(g->gkeys);
    dfree(g->gvals);
    dfree(g->occ);
    dfree(g->occ_n);
    dfree(g->gactive);
    dfree(g->gchanged);
    dfree(g->gbest);
    g->gbest = nullptr;
    dfree(g->gmaj);
    g->gmaj = nullptr;
    g->chunk_g = nullptr;
    g->chunk_e0 = g->chunk_e1 = g->table_off = nullptr;
    g->gkeys = g->occ = g->occ_n = nullptr;
    g->gvals = nullptr;
    g->gactive = g->gchanged = nullptr;
    g->n_chunks = 0;
    g->bins_built = false;
}

// ---------------------------------------------------------------------------
// multi-GPU exchange (distributed.py): changed labels as (vertex, label)
// pairs, marks as per-rank bitmaps
// ---------------------------------------------------------------------------
// pairs[k] = vertex << 32 | label for every own row whose label differs from
// prev (the rank's labels before the sweep); *cnt = number of pairs
// (warp-aggregated atomics; pair order is arbitrary, vertices are unique)
__global__ void k_pack_changed(const int32_t *__restrict__ lab, const int32_t *__restrict__ prev, int64_t row_begin,
                               int64_t n, long long *pairs, unsigned long long *cnt) {
    const int lane = threadIdx.x & 31;
    for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n; base += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = base + threadIdx.x;
        const int32_t c = r < n ? lab[row_begin + r] : 0;
        const bool ch = r < n && c != prev[r];
        const unsigned m = __ballot_sync(0xFFFFFFFFu, ch);
        if (!m) continue;
        unsigned long long pos = 0;
        if (lane == 0) pos = atomicAdd(cnt, (unsigned long long)__popc(m));
        pos = __shfl_sync(0xFFFFFFFFu, pos, 0) + __popc(m & ((1u << lane) - 1));
        if (ch) pairs[pos] = (long long)(((uint64_t)(row_begin + r) << 32) | (uint32_t)c);
    }
}
// lab[vertex] = label for every pair (pairs < 0 are padding)
__global__ void k_apply_pairs(int32_t *lab, const long long *__restrict__ pairs, int64_t n) {
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
        const long long p = pairs[k];
        if (p >= 0) lab[(int64_t)((uint64_t)p >> 32)] = (int32_t)(uint32_t)p;
    }
}
// bits[q][w] bit t = flags[bounds[q] + 32w + t] for every rank range q
// (words words per range); afterwards the flags outside [own_b, own_e) are
// cleared (each rank keeps only its own rows' marks)
__global__ void k_pack_flag_bits(uint8_t *flags, const int64_t *__restrict__ bounds, int P, int64_t words,
                                 uint32_t *bits, int64_t own_b, int64_t own_e) {
    const int64_t tot = (int64_t)P * words;
    for (int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; k < tot; k += (int64_t)gridDim.x * blockDim.x) {
        const int q = (int)(k / words);
        const int64_t w = k - (int64_t)q * words, b = bounds[q], e = bounds[q + 1];
        uint32_t x = 0;
        for (int t = 0; t < 32; ++t) {
            const int64_t i = b + 32 * w + t;
            if (i < e && flags[i]) x |= 1u << t;
        }
        bits[k] = x;
    }
}
__global__ void k_clear_remote_flags(uint8_t *flags, int64_t n, int64_t own_b, int64_t own_e) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        if (i < own_b || i >= own_e) flags[i] = 0;
}
// flags[own_b + i] = OR over the P ranks' bitmaps of the own range
__global__ void k_or_flag_bits(uint8_t *flags, const uint32_t *__restrict__ bits, int P, int64_t words, int64_t own_b,
                               int64_t own_e) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; own_b + i < own_e; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t x = 0;
        for (int q = 0; q < P; ++q) x |= bits[(int64_t)q * words + (i >> 5)];
        flags[own_b + i] = (x >> (i & 31)) & 1u;
    }
}

// Algorithm 1's stop test on the device (nulpa_run's CUDA-graph loop,
// PAPER.md:305-318): iteration l = lv[0] has just swept with Pick-Less lv[1]
// and left its counters in `scratch`; they move to counter slot l; stop
// (conditional = 0) when not Pick-Less and dN/N < tau or l + 1 = maxit,
// else advance l and the Pick-Less flag of iteration l + 1.
// lv: [0] iteration, [1] Pick-Less flag, [2] converged, [3] iterations done.
__global__ void k_loop_step(unsigned long long *scratch, unsigned long long *ctr_all, int32_t *lv, double n_global,
                            double tol, int rho, int maxit, cudaGraphConditionalHandle cond) {
    const int l = lv[0];
    for (int k = threadIdx.x; k < kCtr; k += blockDim.x) ctr_all[(size_t)l * kCtr + k] = scratch[k];
    if (threadIdx.x == 0) {
        const bool pl = lv[1] != 0;
        const bool conv = !pl && (double)scratch[0] / n_global < tol;
        const bool stop = conv || l + 1 >= maxit;
        lv[2] = conv ? 1 : 0;
        lv[3] = l + 1;
        if (!stop) {
            lv[0] = l + 1;
            lv[1] = rho > 0 && (l + 1) % rho == 0;
        }
        cudaGraphSetConditional(cond, stop ? 0u : 1u);
    }
}

__global__ void k_fill_i32(int32_t *p, int64_t n, int32_t v) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) p[i] = v;
}

int grid_for(int64_t n, int threads, int cap_blocks = 0) {
    int64_t b = (n + threads - 1) / threads;
    if (cap_blocks > 0 && b > cap_blocks) b = cap_blocks;
    return (int)std::max<int64_t>(b, 1);
}

// Row a1: the degree-binned frontier.
int build_bins(nulpa_graph *g, int32_t t1, int32_t t2, int32_t t3) {
    free_bins(g);
    g->t1 = t1;
    g->t2 = t2;
    g->t3 = t3;
    const int64_t n = g->n_rows;
    const int64_t per = (int64_t)kBinTile * kBinTiles;
    const int64_t nb = (n + per - 1) / per;
    int64_t *counts = nullptr, *totals = nullptr;
    unsigned long long *edges = nullptr;
    CHECK(dalloc(&counts, (size_t)std::max<int64_t>(nb, 1) * 4));
    CHECK(dalloc(&totals, 4));
    CHECK(dalloc(&edges, 8));
    CU(cudaMemsetAsync(edges, 0, 8 * sizeof(unsigned long long), g->stream));
    if (nb > 0) {
        k_bin_count<<<(unsigned)nb, kBinTile, 0, g->stream>>>(g->offsets, n, t1, t2, t3, counts, edges, edges + 4);
        CU(cudaGetLastError());
        k_bin_scan<<<1, 1024, 0, g->stream>>>(counts, nb, totals);
        CU(cudaGetLastError());
    } else {
        CU(cudaMemsetAsync(totals, 0, 4 * sizeof(int64_t), g->stream));
    }
    int64_t ht[4];
    unsigned long long he[8];
    CU(cudaMemcpyAsync(ht, totals, sizeof ht, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaMemcpyAsync(he, edges, sizeof he, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    {
        const size_t nwmax = (size_t)num_sms() * kWarpCtasPerSm * kWarpWarps;
        CHECK(dalloc(&g->wranges, nwmax));
        CU(cudaMemsetAsync(g->wranges, 0, nwmax * sizeof(unsigned long long), g->stream));   // all ranges empty
    }
    BinLists L;
    for (int b = 0; b < 4; ++b) {
        g->bin_n[b] = ht[b];
        g->bin_e[b] = (int64_t)he[b];
        g->bin_maxdeg[b] = (int64_t)he[4 + b];
        CHECK(dalloc(&g->bin_list[b], (size_t)ht[b]));
        L.l[b] = g->bin_list[b];
    }
    // thread-bin compacted frontier (bulk bins of low degree; allocated here,
    // not in the sweep, which the device loop captures into a CUDA graph)
    if (2 * g->bin_e[0] >= g->M && g->bin_maxdeg[0] <= 8) CHECK(dalloc(&g->trows, (size_t)g->bin_n[0]));
    if (nb > 0) {
        k_bin_scatter<<<(unsigned)nb, kBinTile, 0, g->stream>>>(g->offsets, n, t1, t2, t3, counts, L);
        CU(cudaGetLastError());
    }
    // giant chunks (host-side bookkeeping over the few giant vertices)
    const int64_t ng = g->bin_n[3];
    if (ng > 0) {
        int64_t *ddeg = nullptr;
        CHECK(dalloc(&ddeg, (size_t)(2 * ng)));   // [degrees | row offsets]
        k_gather_degrees<<<grid_for(ng, 256), 256, 0, g->stream>>>(g->offsets, g->bin_list[3], ng, ddeg);
        CU(cudaGetLastError());
        std::vector<int64_t> deg(ng);
        std::vector<int32_t> rows(ng);
        CU(cudaMemcpyAsync(deg.data(), ddeg, ng * sizeof(int64_t), cudaMemcpyDeviceToHost, g->stream));
        CU(cudaMemcpyAsync(rows.data(), g->bin_list[3], ng * sizeof(int32_t), cudaMemcpyDeviceToHost, g->stream));
        std::vector<int64_t> roff(ng);
        CU(cudaMemcpyAsync(roff.data(), ddeg + ng, ng * sizeof(int64_t), cudaMemcpyDeviceToHost, g->stream));
        CU(cudaStreamSynchronize(g->stream));
        dfree(ddeg);
        std::vector<int32_t> cg;
        std::vector<int64_t> c0, c1, toff(ng);
        int64_t slots = 0;
        for (int64_t k = 0; k < ng; ++k) {
            toff[k] = slots;
            slots += capacity_p1((uint32_t)deg[k]) + 1;
            for (int64_t e = 0; e < deg[k]; e += kGiantChunk) {
                cg.push_back((int32_t)k);
                c0.push_back(roff[k] + e);
                c1.push_back(roff[k] + std::min<int64_t>(deg[k], e + kGiantChunk));
            }
        }
        g->n_chunks = (int64_t)cg.size();
        CHECK(dalloc(&g->chunk_g, cg.size()));
        CHECK(dalloc(&g->chunk_e0, c0.size()));
        CHECK(dalloc(&g->chunk_e1, c1.size()));
        CHECK(dalloc(&g->table_off, (size_t)ng));
        CHECK(dalloc(&g->gkeys, (size_t)slots));
        CHECK(dalloc(&g->gvals, (size_t)slots));
        CHECK(dalloc(&g->occ, (size_t)slots));
        CHECK(dalloc(&g->occ_n, (size_t)ng));
        CHECK(dalloc(&g->gactive, (size_t)ng));
        CHECK(dalloc(&g->gchanged, (size_t)ng));
        CHECK(dalloc(&g->gbest, (size_t)ng));
        CHECK(dalloc(&g->gmaj, (size_t)(3 * ng)));
        // on the handle's stream (every bin kernel is ordered after the
        // cudaStreamSynchronize(g->stream) below; the host vectors outlive it)
        CU(cudaMemcpyAsync(g->chunk_g, cg.data(), cg.size() * sizeof(int32_t), cudaMemcpyHostToDevice, g->stream));
        CU(cudaMemcpyAsync(g->chunk_e0, c0.data(), c0.size() * sizeof(int64_t), cudaMemcpyHostToDevice, g->stream));
        CU(cudaMemcpyAsync(g->chunk_e1, c1.data(), c1.size() * sizeof(int64_t), cudaMemcpyHostToDevice, g->stream));
        CU(cudaMemcpyAsync(g->table_off, toff.data(), toff.size() * sizeof(int64_t), cudaMemcpyHostToDevice, g->stream));
        k_fill_i32<<<grid_for(slots, 256, 4096), 256, 0, g->stream>>>(g->gkeys, slots, kEmpty);
        CU(cudaGetLastError());
        CU(cudaMemsetAsync(g->gvals, 0, slots * sizeof(float), g->stream));
        CU(cudaMemsetAsync(g->occ_n, 0, ng * sizeof(int32_t), g->stream));
        CU(cudaStreamSynchronize(g->stream));          // before cg / c0 / c1 / toff go out of scope
    }
    CU(cudaStreamSynchronize(g->stream));
    {
        // ID locality from <= 65536 sampled rows (reuses `edges` as the accumulator)
        const int64_t ns = std::min<int64_t>(n, 65536), step = ns ? n / ns : 1;
        unsigned long long h[2] = {0, 0};
        if (ns > 0) {
            CU(cudaMemsetAsync(edges, 0, 2 * sizeof(unsigned long long), g->stream));
            k_locality<<<grid_for(ns, 256), 256, 0, g->stream>>>(g->offsets, g->indices, g->row_begin, step, ns, edges);
            CU(cudaGetLastError());
            CU(cudaMemcpyAsync(h, edges, sizeof h, cudaMemcpyDeviceToHost, g->stream));
            CU(cudaStreamSynchronize(g->stream));
        }
        g->locality = h[0] ? (double)h[1] / (double)h[0] : 0.0;
    }
    dfree(counts);
    dfree(totals);
    dfree(edges);
    for (int b = 0; b < 4; ++b) {
        g->stats.bin_vertices[b] = g->bin_n[b];
        g->stats.bin_edges[b] = g->bin_e[b];
    }
    g->bins_built = true;
    return NULPA_OK;
}

int validate_params(const nulpa_params &p) {
    if (!(p.tolerance >= 0.0)) return fail(NULPA_EINVAL, "tolerance must be >= 0");
    if (p.max_iterations < 0) return fail(NULPA_EINVAL, "max_iterations must be >= 0");
    if (p.mode != NULPA_ASYNC && p.mode != NULPA_SYNC) return fail(NULPA_EINVAL, "mode must be NULPA_ASYNC or NULPA_SYNC");
    if (p.switch_degree < 1 || p.switch_degree > 33)
        return fail(NULPA_EINVAL, "switch_degree must be in [1, 33] (thread-per-vertex tables live in registers)");
    if (p.block_degree < p.switch_degree || p.block_degree > 256)
        return fail(NULPA_EINVAL, "block_degree must be in [switch_degree, 256] (warp tables hold 255 slots)");
    if (p.tie_rule != NULPA_TIE_SMALLEST) return fail(NULPA_EINVAL, "tie_rule must be NULPA_TIE_SMALLEST (0): ties go to the smallest label (R6)");
    if (p.bin_order < 0 || p.bin_order > 4) return fail(NULPA_EINVAL, "bin_order must be 0, 1, 2, 3 or 4");
    if (p.first_sweep_block < 0 || p.first_sweep_block > 1024 || p.sweep_block < 0 || p.sweep_block > 1024)
        return fail(NULPA_EINVAL, "first_sweep_block and sweep_block must be in [0, 1024]");
    if (p.wide_degree < 1 || p.wide_degree > 1024)   // distinct labels <= D <= 1023 = p1 (R5 always finds a slot)
        return fail(NULPA_EINVAL, "wide_degree must be in [1, 1024] (wide warp tables hold 1023 slots)");
    if (p.giant_degree < p.block_degree || p.giant_degree > 4096)
        return fail(NULPA_EINVAL, "giant_degree must be in [block_degree, 4096] (CTA tables hold 4095 slots)");
    return NULPA_OK;
}

int ensure_bins(nulpa_graph *g, const nulpa_params &p) {
    if (g->bins_built && g->t1 == p.switch_degree && g->t2 == p.block_degree && g->t3 == p.giant_degree) return NULPA_OK;
    return build_bins(g, p.switch_degree, p.block_degree, p.giant_degree);
}

// The thread bin in kThreadWaves launches over consecutive slices of the
// bin list (asynchronous mode, when the thread bin holds at least half of
// the CSR entries and spans fewer than kThreadWaves grid-stride steps): a
// vertex of slice w sees the labels slices
// < w wrote in this sweep, so on graphs whose neighbours have unrelated IDs
// (k-mer paths, permuted IDs) about half of its neighbours are already
// updated, as in the sequential ID-order sweep of Algorithm 1 -- one launch
// over a small bin processes every vertex at once (Jacobi) and lands ~0.02
// below the sequential sweep's modularity on k-mer graphs.
#ifndef NULPA_THREAD_WAVES
#define NULPA_THREAD_WAVES 8
#endif
constexpr int kThreadWaves = NULPA_THREAD_WAVES;
static_assert(kThreadWaves <= kCtr - kCtrTScan, "one compaction counter per wave");
#ifndef NULPA_TACT_V8
#define NULPA_TACT_V8 4                  // k_tact rows in flight together for degrees 5..8 (k-mer 3.93e9 edges/s; 2 rows: 3.79e9)
#endif
#ifndef NULPA_TCOMPACT
#define NULPA_TCOMPACT 1                 // asynchronous bulk thread bins: compacted frontier
#endif
template <bool SYNC, bool W>
int launch_thread_bin(nulpa_graph *g, const SweepArgs &a, cudaStream_t st) {
    const int64_t n = g->bin_n[0];
    const int64_t md = g->bin_maxdeg[0];     // register table sized by the bin's largest degree
    // a bin spanning >= kThreadWaves grid-stride steps is already swept in
    // order (step s of every thread covers entries [4Ts, 4T(s+1))): one launch
    const int64_t per_step = 4LL * kThreadThreads * num_sms() * 8;
    // order matters for the sweep's result only where the thread bin is most
    // of the graph (path-like k-mer / road graphs); elsewhere a thin bin of
    // low-degree vertices is one launch
    const bool bulk = 2 * g->bin_e[0] >= g->M;
    int64_t waves = SYNC || !bulk ? 1 : (kThreadWaves * per_step + n - 1) / std::max<int64_t>(n, 1);
    waves = std::max<int64_t>(1, std::min<int64_t>({waves, (int64_t)kThreadWaves, n / 1024}));
    // asynchronous bulk bins of low degree: compacted frontier (k_tscan + k_tact)
    const bool compact = NULPA_TCOMPACT && !SYNC && bulk && md <= 8;
    if (compact && !g->trows) return fail(NULPA_ESTATE, "thread-bin frontier not allocated");
    for (int64_t w = 0; w < waves; ++w) {
        // slice bounds on multiples of 4 entries (k_thread reads the list 16 bytes at a time)
        const int64_t b0 = (n * w / waves) & ~INT64_C(3), b1 = w + 1 == waves ? n : (n * (w + 1) / waves) & ~INT64_C(3);
        const int64_t m = b1 - b0;
        const int32_t *list = g->bin_list[0] + b0;
        const int grid = bulk ? grid_for((m + 3) / 4, kThreadThreads, num_sms() * 8)   // 4 entries per thread and step
                              : grid_for(m, kThreadThreads, num_sms() * 32);
        if (compact) {
            unsigned long long *cnt = a.ctr + kCtrTScan + w;
            k_tscan<<<grid_for(m, 4 * kTScanThreads, num_sms() * 8), kTScanThreads, 0, st>>>(a, list, m, g->trows, cnt);
            if (md <= 4)
                k_tact<W, 4, 4><<<grid, kThreadThreads, 0, st>>>(a, g->trows, cnt);
            else
                k_tact<W, 8, NULPA_TACT_V8><<<grid, kThreadThreads, 0, st>>>(a, g->trows, cnt);
            CU(cudaGetLastError());
            continue;
        }
        if (md <= 4)
            k_thread<SYNC, W, 4><<<grid, kThreadThreads, 0, st>>>(a, list, m, bulk);
        else if (md <= 8)
            k_thread<SYNC, W, 8><<<grid, kThreadThreads, 0, st>>>(a, list, m, bulk);
        else if (md <= 16)
            k_thread<SYNC, W, 16><<<grid, kThreadThreads, 0, st>>>(a, list, m, bulk);
        else
            k_thread<SYNC, W, 32><<<grid, kThreadThreads, 0, st>>>(a, list, m, bulk);
        CU(cudaGetLastError());
    }
    g->stats.launches[0] += (int)waves * (compact ? 2 : 1) - 1;
    return NULPA_OK;
}

template <bool SYNC, bool W>
int sweep_impl(nulpa_graph *g, int pickless, const nulpa_params &p, unsigned long long *ctr, bool timing, int slot,
               const int32_t *pl_dev) {
    SweepArgs a;
    a.pl_dev = pl_dev;
    a.first = g->sweeps_since_reset == 0;
    a.kbits = 1;
    while (a.kbits < 31 && (INT64_C(1) << a.kbits) <= g->n_global) ++a.kbits;   // key + 1 <= n_global < 2^kbits
    a.offsets = g->offsets;
    a.indices = g->indices;
    a.weights = g->weights;
    a.row_begin = g->row_begin;
    a.pickless = pickless;
    const int sched_block = g->sweeps_since_reset == 0 ? p.first_sweep_block : p.sweep_block;
    a.ctr = ctr;
    if (SYNC) {
        CU(cudaMemcpyAsync(g->labels_prev, g->labels, g->n_global * sizeof(int32_t), cudaMemcpyDeviceToDevice, g->stream));
        CU(cudaMemcpyAsync(g->flags_prev, g->flags, g->n_global, cudaMemcpyDeviceToDevice, g->stream));
        CU(cudaMemsetAsync(g->flags, 0, g->n_global, g->stream));
        a.lab_in = g->labels_prev;
        a.flag_in = g->flags_prev;
        g->stats.other_launches += 3;
    } else {
        a.lab_in = g->labels;
        a.flag_in = g->flags;
    }
    a.lab_out = g->labels;
    a.flag_out = g->flags;
    const int sms = num_sms();
    const bool o32 = g->M + 64 < (INT64_C(1) << 32);  // 32-bit row addressing in k_warp
    cudaStream_t cs = g->stream;                  // stream of the bin being launched
    auto rec = [&](int b, int which) -> int {
        if (timing) CU(cudaEventRecord(g->ev[(slot * 4 + b) * 2 + which], cs));
        return NULPA_OK;
    };
    auto run_giant = [&]() -> int {
        const int64_t ng = g->bin_n[3];
        CHECK(rec(3, 0));
        if (ng > 0) {
            GiantArgs ga;
            ga.verts = g->bin_list[3];
            ga.chunk_g = g->chunk_g;
            ga.chunk_e0 = g->chunk_e0;
            ga.chunk_e1 = g->chunk_e1;
            ga.table_off = g->table_off;
            ga.keys = g->gkeys;
            ga.vals = g->gvals;
            ga.occ = g->occ;
            ga.occ_n = g->occ_n;
            ga.active = g->gactive;
            ga.changed = g->gchanged;
            ga.best = g->gbest;
            ga.maj = g->gmaj;
            const size_t smem = kGiantCap * (sizeof(int32_t) + sizeof(float)) + kGiantChunk * sizeof(uint16_t);
            // set on every launch: the attribute is per device, the handle may live on any
            CU(cudaFuncSetAttribute(k_giant_accumulate<SYNC, W>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
            k_giant_snapshot<SYNC><<<grid_for(ng, 256), 256, 0, cs>>>(a, ga, ng);
#if NULPA_MAJORITY
            if (!a.first) {
                k_giant_count<W><<<(unsigned)g->n_chunks, kBlockThreads, 0, cs>>>(a, ga);
                g->stats.launches[3] += 1;
            }
#endif
            k_giant_accumulate<SYNC, W><<<(unsigned)g->n_chunks, kBlockThreads, smem, cs>>>(a, ga);
            k_giant_decide<SYNC><<<grid_for(ng, 128), 128, 0, cs>>>(a, ga, ng);
            k_giant_finish<<<(unsigned)g->n_chunks, kBlockThreads, 0, cs>>>(a, ga);
            CU(cudaGetLastError());
            g->stats.launches[3] += 4;
        }
        CHECK(rec(3, 1));
        return NULPA_OK;
    };
    auto run_block = [&]() -> int {
        const int64_t n = g->bin_n[2];
        CHECK(rec(2, 0));
        if (n > 0) {
            // frontier split at wide_degree: warp-per-vertex (1023-slot tables) below, CTA-per-vertex above
            if (!g->brecs) CHECK(dalloc(reinterpret_cast<VRec **>(&g->brecs), (size_t)(2 * n)));
            VRec *rw = reinterpret_cast<VRec *>(g->brecs), *rb = rw + n;
            // k_block: table of the largest p1, two TMA row buffers
            auto launch_block = [&](auto kern, int nt, int maxdeg, const VRec *recs_b, unsigned long long *cnt) -> int {
                const int cap = (int)capacity_p1((uint32_t)maxdeg) + 1;
                const int rowcap = (maxdeg + 4 + 3) & ~3;
                const size_t smem = (size_t)cap * (NULPA_BLOCK_LIST ? 16 : 12) + (size_t)rowcap * 4 * 2 * (W ? 2 : 1);
                CU(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                int per_sm = 0;
                CU(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, nt, smem));
                kern<<<grid_for(n, 1, sms * std::max(1, per_sm)), nt, smem, cs>>>(a, recs_b, cnt, cap, rowcap);
                CU(cudaGetLastError());
                return NULPA_OK;
            };
            const uint32_t split = (uint32_t)std::max(p.wide_degree, p.block_degree);
            k_frontier<SYNC><<<grid_for(n, kFrontTile, sms * 8), kFrontThreads, 0, cs>>>(a, g->bin_list[2], n, 2, rw, ctr + kCtrRecsW,
                                                                          split, rb, ctr + kCtrRecsB);
            if (split > (uint32_t)p.block_degree && NULPA_WIDE_TMA) {
                // degree < split (<= 1023): k_block with 4 warps per vertex, 1023-slot
                // tables and 1 KB row buffers -- many vertices in flight per SM
                const int md = (int)split - 1;
                if (md + 3 <= 4 * 128)
                    CHECK(launch_block(k_block<SYNC, W, 4, 128>, 128, md, rw, ctr + kCtrRecsW));
                else
                    CHECK(launch_block(k_block<SYNC, W, 8, 128>, 128, md, rw, ctr + kCtrRecsW));
                g->stats.launches[2] += 1;
            } else if (split > (uint32_t)p.block_degree) {
                const WarpSched ws{SCHED_GUIDED, NULPA_WIDE_K, ctr + kCtrSchedB, nullptr};
                if (o32)
                    k_warp<SYNC, W, kWideSlots, true><<<sms * kWideCtasPerSm, kWideWarps * 32, 0, cs>>>(a, rw, ctr + kCtrRecsW, 2, ws);
                else
                    k_warp<SYNC, W, kWideSlots, false><<<sms * kWideCtasPerSm, kWideWarps * 32, 0, cs>>>(a, rw, ctr + kCtrRecsW, 2, ws);
                g->stats.launches[2] += 1;
            }
            const int maxdeg = std::max(1, p.giant_degree - 1);
            if (maxdeg + 3 <= 8 * kBlkThreads) CHECK(launch_block(k_block<SYNC, W, 8, kBlkThreads>, kBlkThreads, maxdeg, rb, ctr + kCtrRecsB));
            else CHECK(launch_block(k_block<SYNC, W, 16, kBlkThreads>, kBlkThreads, maxdeg, rb, ctr + kCtrRecsB));
            g->stats.launches[2] += 2;
        }
        CHECK(rec(2, 1));
        return NULPA_OK;
    };
    // bin_order 4 (auto): 3 when the warp bin holds >= 2/3 of the CSR entries
    // (web, SBM: the block + giant bins fill its tail), else 1 (social graphs:
    // block + giant bins are ~half the entries and would wait for the warp
    // bin's CTAs on the low-priority stream; measured R-MAT 4M/70M 17.0 ->
    // 19.8e9 edges/s with 1)
    const int order = p.bin_order == 4 ? (3 * g->bin_e[1] >= 2 * g->M ? 3 : 1) : p.bin_order;
    bool mid_fork = false;                        // bin_order 3: record ev_mid after the warp-bin frontier
    auto run_warp = [&]() -> int {
        const int64_t n = g->bin_n[1];
        CHECK(rec(1, 0));
        if (n > 0) {
            if (!g->wrecs) CHECK(dalloc(reinterpret_cast<VRec **>(&g->wrecs), (size_t)n));
            VRec *recs = reinterpret_cast<VRec *>(g->wrecs);
            k_frontier<SYNC><<<grid_for(n, kFrontTile, sms * 8), kFrontThreads, 0, cs>>>(a, g->bin_list[1], n, 1, recs, ctr + kCtrRecs,
                                                                          0xFFFFFFFFu, nullptr, nullptr);
            if (mid_fork) CU(cudaEventRecord(g->ev_mid, cs));
            WarpSched ws{sched_block == 0 ? SCHED_STEAL : sched_block == 1 ? SCHED_STRIDED : SCHED_GUIDED,
                         sched_block, ctr + kCtrSchedW, g->wranges};
            int grid = sms * kWarpCtasPerSm;
            if (ws.mode == SCHED_STEAL && g->locality >= kLocalRuns) {
                // each warp walks one run of bin / warps rows; on a small bin
                // (a test graph, a row shard of a multi-GPU run) whose IDs
                // carry locality (web crawls in URL order, road networks)
                // launch only enough warps for runs of >= kMinFirstRun rows
                // (modularity: labels propagate along ID order within a run;
                // DESIGN.md "Quality notes").  Without ID locality (permuted
                // SBM / R-MAT IDs) runs buy nothing: full grid.
                ws.K = (int)(kMinFirstRun / 32);
                const int64_t warps = std::max<int64_t>(1, n / kMinFirstRun);
                grid = (int)std::min<int64_t>(grid, (warps + kWarpWarps - 1) / kWarpWarps);
            }
            if (o32)
                k_warp<SYNC, W, kWarpSlots, true><<<grid, kWarpWarps * 32, 0, cs>>>(a, recs, ctr + kCtrRecs, 1, ws);
            else
                k_warp<SYNC, W, kWarpSlots, false><<<grid, kWarpWarps * 32, 0, cs>>>(a, recs, ctr + kCtrRecs, 1, ws);
            CU(cudaGetLastError());
            g->stats.launches[1] += 2;
        }
        CHECK(rec(1, 1));
        return NULPA_OK;
    };
    auto run_thread = [&]() -> int {
        const int64_t n = g->bin_n[0];
        CHECK(rec(0, 0));
        if (n > 0) {
            CHECK((launch_thread_bin<SYNC, W>(g, a, cs)));
            g->stats.launches[0] += 1;
        }
        CHECK(rec(0, 1));
        return NULPA_OK;
    };
    if (order == 0) {
        CHECK(run_giant());
        CHECK(run_block());
        CHECK(run_warp());
        CHECK(run_thread());
    } else if (order == 3) {
        // thread bin on the caller's stream; warp bin on a high-priority
        // stream; block + giant bins on a low-priority side stream released
        // after the warp-bin frontier: k_warp's CTAs take every SM's register
        // file first, the side kernels' CTAs fill SMs as warp-bin CTAs retire
        // (the warp bin's tail) -- asynchronous reads of concurrently written
        // labels are what the asynchronous sweep already does
        if (!g->hi) {
            int least = 0, greatest = 0;
            CU(cudaDeviceGetStreamPriorityRange(&least, &greatest));
            CU(cudaStreamCreateWithPriority(&g->hi, cudaStreamNonBlocking, greatest));
            if (!g->side) CU(cudaStreamCreateWithPriority(&g->side, cudaStreamNonBlocking, least));
            if (!g->ev_fork) CU(cudaEventCreateWithFlags(&g->ev_fork, cudaEventDisableTiming));
            if (!g->ev_join) CU(cudaEventCreateWithFlags(&g->ev_join, cudaEventDisableTiming));
            CU(cudaEventCreateWithFlags(&g->ev_mid, cudaEventDisableTiming));
            CU(cudaEventCreateWithFlags(&g->ev_join2, cudaEventDisableTiming));
        }
        CHECK(run_thread());
        CU(cudaEventRecord(g->ev_fork, g->stream));
        CU(cudaStreamWaitEvent(g->hi, g->ev_fork, 0));
        CU(cudaEventRecord(g->ev_mid, g->hi));          // (re-recorded after the frontier if the bin is non-empty)
        cs = g->hi;
        mid_fork = true;
        CHECK(run_warp());
        CU(cudaEventRecord(g->ev_join, g->hi));
        CU(cudaStreamWaitEvent(g->side, g->ev_mid, 0));
        cs = g->side;
        CHECK(run_block());
        CHECK(run_giant());
        CU(cudaEventRecord(g->ev_join2, g->side));
        cs = g->stream;
        CU(cudaStreamWaitEvent(g->stream, g->ev_join, 0));
        CU(cudaStreamWaitEvent(g->stream, g->ev_join2, 0));
    } else if (order == 2) {
        // block + giant bins on a side stream, concurrent with thread + warp:
        // their latency-bound CTAs fill the SMs the warp bin leaves idle
        if (!g->side) {
            CU(cudaStreamCreateWithFlags(&g->side, cudaStreamNonBlocking));
            CU(cudaEventCreateWithFlags(&g->ev_fork, cudaEventDisableTiming));
            CU(cudaEventCreateWithFlags(&g->ev_join, cudaEventDisableTiming));
        }
        CU(cudaEventRecord(g->ev_fork, g->stream));
        CU(cudaStreamWaitEvent(g->side, g->ev_fork, 0));
        cs = g->side;
        CHECK(run_block());
        CHECK(run_giant());
        CU(cudaEventRecord(g->ev_join, g->side));
        cs = g->stream;
        CHECK(run_thread());
        CHECK(run_warp());
        CU(cudaStreamWaitEvent(g->stream, g->ev_join, 0));
    } else {
        CHECK(run_thread());
        CHECK(run_warp());
        CHECK(run_block());
        CHECK(run_giant());
    }
    return NULPA_OK;
}

int sweep(nulpa_graph *g, int pickless, const nulpa_params &p, unsigned long long *ctr, bool timing, int slot,
          const int32_t *pl_dev = nullptr) {
    const bool w = g->weights != nullptr;
    if (p.mode == NULPA_SYNC && !g->labels_prev) {
        CHECK(dalloc(&g->labels_prev, (size_t)g->n_global));
        CHECK(dalloc(&g->flags_prev, (size_t)g->n_global));
    }
    const int sel = (p.mode == NULPA_SYNC ? 2 : 0) + (w ? 1 : 0);
    int r;
    switch (sel) {
    case 0: r = sweep_impl<false, false>(g, pickless, p, ctr, timing, slot, pl_dev); break;
    case 1: r = sweep_impl<false, true>(g, pickless, p, ctr, timing, slot, pl_dev); break;
    case 2: r = sweep_impl<true, false>(g, pickless, p, ctr, timing, slot, pl_dev); break;
    default: r = sweep_impl<true, true>(g, pickless, p, ctr, timing, slot, pl_dev); break;
    }
    ++g->sweeps_since_reset;
    return r;
}

bool same_loop_params(const nulpa_params &a, const nulpa_params &b) {
    return a.tolerance == b.tolerance && a.max_iterations == b.max_iterations && a.pickless_period == b.pickless_period &&
           a.mode == b.mode && a.switch_degree == b.switch_degree && a.block_degree == b.block_degree &&
           a.giant_degree == b.giant_degree && a.bin_order == b.bin_order && a.wide_degree == b.wide_degree &&
           a.sweep_block == b.sweep_block;
}

// The device loop: graph = [k_loop_step for sweep 0] -> while (cond) {
// memset(scratch counters); sweep (Pick-Less flag from loopvars[1], bins
// as in a host-loop sweep >= 1); k_loop_step }.  Captured from the handle's
// stream (the bin streams join the capture through their events).
int build_loop(nulpa_graph *g, const nulpa_params &p, int maxit) {
    free_loop(g);
    if (!g->loopvars) CHECK(dalloc(&g->loopvars, 4));
    unsigned long long *scratch = g->ctr + (size_t)kMaxIter * kCtr;
    CU(cudaGraphCreate(&g->loop_graph, 0));
    cudaGraphConditionalHandle cond;
    CU(cudaGraphConditionalHandleCreate(&cond, g->loop_graph, 1, cudaGraphCondAssignDefault));
    // first node: the stop test of sweep 0 (launched before the graph)
    cudaGraphNode_t first;
    {
        cudaKernelNodeParams kp = {};
        double n_global = (double)g->n_global, tol = p.tolerance;
        int rho = p.pickless_period;
        unsigned long long *ctr_all = g->ctr;
        int32_t *lv = g->loopvars;
        void *args[] = {&scratch, &ctr_all, &lv, &n_global, &tol, &rho, &maxit, &cond};
        kp.func = (void *)k_loop_step;
        kp.gridDim = dim3(1);
        kp.blockDim = dim3(32);
        kp.kernelParams = args;
        CU(cudaGraphAddKernelNode(&first, g->loop_graph, nullptr, 0, &kp));
    }
    cudaGraphNodeParams cp = {};
    cp.type = cudaGraphNodeTypeConditional;
    cp.conditional.handle = cond;
    cp.conditional.type = cudaGraphCondTypeWhile;
    cp.conditional.size = 1;
    cudaGraphNode_t wnode;
    CU(cudaGraphAddNode(&wnode, g->loop_graph, &first, 1, &cp));
    cudaGraph_t body = cp.conditional.phGraph_out[0];
    int l0[4];
    memcpy(l0, g->stats.launches, sizeof l0);
    const int o0 = g->stats.other_launches;
    if (!g->cap) CU(cudaStreamCreateWithFlags(&g->cap, cudaStreamNonBlocking));
    cudaStream_t user = g->stream;
    g->stream = g->cap;                                  // the sweep's kernels go to the capture stream
    CU(cudaStreamBeginCaptureToGraph(g->stream, body, nullptr, nullptr, 0, cudaStreamCaptureModeRelaxed));
    int r = NULPA_OK;
    if (cudaMemsetAsync(scratch, 0, kCtr * sizeof(unsigned long long), g->stream) != cudaSuccess) r = NULPA_ECUDA;
    if (r == NULPA_OK) r = sweep(g, 0, p, scratch, false, 0, g->loopvars + 1);
    if (r == NULPA_OK) {
        double n_global = (double)g->n_global;
        k_loop_step<<<1, 32, 0, g->stream>>>(scratch, g->ctr, g->loopvars, n_global, p.tolerance, p.pickless_period, maxit, cond);
        if (cudaGetLastError() != cudaSuccess) r = NULPA_ECUDA;
    }
    cudaGraph_t captured = nullptr;
    const cudaError_t ec = cudaStreamEndCapture(g->stream, &captured);
    g->stream = user;
    if (r != NULPA_OK) return r == NULPA_ECUDA ? fail(NULPA_ECUDA, "capturing the device loop failed") : r;
    CU(ec);
    for (int b = 0; b < 4; ++b) {
        g->loop_launches[b] = g->stats.launches[b] - l0[b];
        g->stats.launches[b] = l0[b];
    }
    g->loop_other = g->stats.other_launches - o0 + 2;          // + the two k_loop_step launches' bookkeeping
    g->stats.other_launches = o0;
    CU(cudaGraphInstantiate(&g->loop_exec, g->loop_graph, 0));
    g->loop_p = p;
    return NULPA_OK;
}

int reset_state(nulpa_graph *g) {
    k_init_state<<<grid_for(g->n_global, 256, num_sms() * 16), 256, 0, g->stream>>>(g->labels, g->flags, g->n_global);
    CU(cudaGetLastError());
    g->stats.other_launches += 1;
    g->sweeps_since_reset = 0;
    return NULPA_OK;
}

void zero_stats_counts(nulpa_stats *s) {
    int64_t bv[4], be[4];
    memcpy(bv, s->bin_vertices, sizeof bv);
    memcpy(be, s->bin_edges, sizeof be);
    memset(s, 0, sizeof *s);
    memcpy(s->bin_vertices, bv, sizeof bv);
    memcpy(s->bin_edges, be, sizeof be);
}

int ensure_events(nulpa_graph *g) {
    if (g->events) return NULPA_OK;
    for (auto &e : g->ev) CU(cudaEventCreate(&e));
    CU(cudaEventCreate(&g->ev_run[0]));
    CU(cudaEventCreate(&g->ev_run[1]));
    g->events = true;
    return NULPA_OK;
}

int resolve_mem(const void *p, int memkind) {
    if (memkind != NULPA_MEM_HOST && memkind != NULPA_MEM_DEVICE) return fail(NULPA_EINVAL, "memkind must be NULPA_MEM_HOST or NULPA_MEM_DEVICE");
    (void)p;
    return NULPA_OK;
}

// R12: reject weights that are negative, NaN or infinite (the argmax orders
// IEEE bit patterns and the giant bin's running maximum needs totals that
// only grow).  One device pass over the weights, counted in a spare slot of
// the handle's counters.
int check_weights(nulpa_graph *g) {
    if (!g->weights || g->M == 0) return NULPA_OK;
    unsigned long long *bad = g->ctr + (size_t)kMaxIter * kCtr + kCtr - 1;
    CU(cudaMemsetAsync(bad, 0, sizeof *bad, g->stream));
    k_check_weights<<<grid_for(g->M, 256, num_sms() * 8), 256, 0, g->stream>>>(g->weights, g->M, bad);
    CU(cudaGetLastError());
    unsigned long long h = 0;
    CU(cudaMemcpyAsync(&h, bad, sizeof h, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    if (h) return fail(NULPA_EINVAL, "%llu weights are negative, NaN or infinite (weights must be finite and >= 0, R12)", h);
    return NULPA_OK;
}

// Labels passed in by the caller must be vertex IDs in [0, n_global) (they
// index Sigma in the modularity kernels and the label-keyed tables).
int check_labels(nulpa_graph *g, const int32_t *lab, int memkind) {
    const int64_t n = g->n_global;
    if (memkind == NULPA_MEM_HOST) {
        for (int64_t i = 0; i < n; ++i)
            if (lab[i] < 0 || (int64_t)lab[i] >= n)
                return fail(NULPA_EINVAL, "label %d of vertex %lld is outside [0, %lld)", lab[i], (long long)i, (long long)n);
        return NULPA_OK;
    }
    if (n == 0) return NULPA_OK;
    unsigned long long *bad = g->ctr + (size_t)kMaxIter * kCtr + kCtr - 1;
    CU(cudaMemsetAsync(bad, 0, sizeof *bad, g->stream));
    k_check_labels<<<grid_for(n, 256, num_sms() * 8), 256, 0, g->stream>>>(lab, n, bad);
    CU(cudaGetLastError());
    unsigned long long h = 0;
    CU(cudaMemcpyAsync(&h, bad, sizeof h, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    if (h) return fail(NULPA_EINVAL, "%llu labels are outside [0, %lld)", h, (long long)n);
    return NULPA_OK;
}

}  // namespace

// ---------------------------------------------------------------------------
// C ABI
// ---------------------------------------------------------------------------
extern "C" {

void nulpa_default_params(nulpa_params *p) {
    if (!p) return;
    p->tolerance = 0.05;
    p->max_iterations = 20;
    p->pickless_period = 4;
    p->mode = NULPA_ASYNC;
    p->switch_degree = 16;
    p->block_degree = 256;
    p->giant_degree = 2048;
    p->reset = 1;
    p->timing = 0;
    p->tie_rule = NULPA_TIE_SMALLEST;
    p->bin_order = 4;
    p->wide_degree = 512;
    p->first_sweep_block = 0;
    p->sweep_block = 4;
    p->device_loop = 1;
}

const char *nulpa_last_error(void) { return g_err.c_str(); }

const char *nulpa_version(void) { return "nulpa 0.1.0 sm_100a"; }

int nulpa_create(const int64_t *offsets, const int32_t *indices, const float *weights, int64_t n_rows,
                 int64_t n_global, int64_t row_begin, int memkind, void *stream, nulpa_graph **out) {
    g_err.clear();
    if (!out) return fail(NULPA_EINVAL, "out is NULL");
    *out = nullptr;
    if (!offsets) return fail(NULPA_EINVAL, "offsets is NULL");
    if (n_rows < 0 || n_global < 0 || row_begin < 0 || row_begin + n_rows > n_global)
        return fail(NULPA_EINVAL, "need 0 <= row_begin, row_begin + n_rows <= n_global");
    if (n_global > INT32_MAX) return fail(NULPA_EINVAL, "n_global must fit int32 vertex IDs");
    CHECK(resolve_mem(offsets, memkind));
    nulpa_graph *g = new nulpa_graph();
    memset(&g->stats, 0, sizeof g->stats);
    g->n_rows = n_rows;
    g->n_global = n_global;
    g->row_begin = row_begin;
    g->stream = (cudaStream_t)stream;
    auto bail = [&](int code) {
        nulpa_destroy(g);
        return code;
    };
    int64_t M = 0;
    if (memkind == NULPA_MEM_HOST) {
        M = offsets[n_rows];
        if (offsets[0] != 0) return bail(fail(NULPA_EINVAL, "offsets[0] must be 0"));
    } else {
        int64_t o0 = 0;
        cudaError_t e = cudaMemcpy(&M, offsets + n_rows, sizeof M, cudaMemcpyDeviceToHost);
        if (e == cudaSuccess) e = cudaMemcpy(&o0, offsets, sizeof o0, cudaMemcpyDeviceToHost);
        if (e != cudaSuccess) return bail(fail(NULPA_ECUDA, "reading device offsets failed: %s", cudaGetErrorString(e)));
        if (o0 != 0) return bail(fail(NULPA_EINVAL, "offsets[0] must be 0"));
    }
    if (M < 0) return bail(fail(NULPA_EINVAL, "offsets[n_rows] must be >= 0"));
    if (M > 0 && !indices) return bail(fail(NULPA_EINVAL, "indices is NULL"));
    if (M >= (INT64_C(1) << 48)) return bail(fail(NULPA_EINVAL, "more than 2^48 CSR entries"));
    g->M = M;
    if (memkind == NULPA_MEM_DEVICE) {
        g->offsets = const_cast<int64_t *>(offsets);
        g->indices = const_cast<int32_t *>(indices);
        g->weights = const_cast<float *>(weights);
        g->own_csr = false;
    } else {
        g->own_csr = true;
        int r;
        if ((r = dalloc(&g->offsets, (size_t)n_rows + 1))) return bail(r);
        if ((r = dalloc(&g->indices, (size_t)M))) return bail(r);
        if (weights && (r = dalloc(&g->weights, (size_t)M))) return bail(r);
        cudaError_t e = cudaMemcpyAsync(g->offsets, offsets, (n_rows + 1) * sizeof(int64_t), cudaMemcpyHostToDevice, g->stream);
        if (e == cudaSuccess && M) e = cudaMemcpyAsync(g->indices, indices, M * sizeof(int32_t), cudaMemcpyHostToDevice, g->stream);
        if (e == cudaSuccess && M && weights) e = cudaMemcpyAsync(g->weights, weights, M * sizeof(float), cudaMemcpyHostToDevice, g->stream);
        if (e != cudaSuccess) return bail(fail(NULPA_ECUDA, "host->device copy failed: %s", cudaGetErrorString(e)));
    }
    int r;
    if ((r = dalloc(&g->own_labels, (size_t)n_global))) return bail(r);
    if ((r = dalloc(&g->own_flags, (size_t)n_global))) return bail(r);
    g->labels = g->own_labels;
    g->flags = g->own_flags;
    if ((r = dalloc(&g->ctr, (size_t)(kMaxIter + 1) * kCtr))) return bail(r);
    if (cudaMallocHost((void **)&g->ctr_host, (kMaxIter + 1) * kCtr * sizeof(unsigned long long)) != cudaSuccess)
        return bail(fail(NULPA_ENOMEM, "cudaMallocHost failed"));
    if ((r = check_weights(g))) return bail(r);
    if ((r = reset_state(g))) return bail(r);
    nulpa_params p;
    nulpa_default_params(&p);
    if ((r = build_bins(g, p.switch_degree, p.block_degree, p.giant_degree))) return bail(r);
    *out = g;
    return NULPA_OK;
}

int nulpa_pack_changed(nulpa_graph *g, const int32_t *prev_device, long long *pairs_device, int64_t *count) {
    if (!g || !prev_device || !pairs_device || !count) return fail(NULPA_EINVAL, "null argument");
    unsigned long long *cnt = g->ctr + (size_t)kMaxIter * kCtr + kCtr - 1;
    CU(cudaMemsetAsync(cnt, 0, sizeof *cnt, g->stream));
    if (g->n_rows > 0) {
        k_pack_changed<<<grid_for(g->n_rows, 256, num_sms() * 8), 256, 0, g->stream>>>(g->labels, prev_device, g->row_begin,
                                                                                     g->n_rows, pairs_device, cnt);
        CU(cudaGetLastError());
    }
    unsigned long long h = 0;
    CU(cudaMemcpyAsync(&h, cnt, sizeof h, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    *count = (int64_t)h;
    return NULPA_OK;
}

int nulpa_apply_pairs(nulpa_graph *g, const long long *pairs_device, int64_t n) {
    if (!g || (n > 0 && !pairs_device)) return fail(NULPA_EINVAL, "null argument");
    if (n > 0) {
        k_apply_pairs<<<grid_for(n, 256, num_sms() * 8), 256, 0, g->stream>>>(g->labels, pairs_device, n);
        CU(cudaGetLastError());
    }
    return NULPA_OK;
}

int nulpa_pack_flag_bits(nulpa_graph *g, const int64_t *bounds_device, int P, int64_t words, uint32_t *bits_device) {
    if (!g || !bounds_device || !bits_device || P < 1 || words < 0) return fail(NULPA_EINVAL, "bad argument");
    const int64_t tot = (int64_t)P * words;
    if (tot > 0) {
        k_pack_flag_bits<<<grid_for(tot, 256, num_sms() * 8), 256, 0, g->stream>>>(g->flags, bounds_device, P, words,
                                                                                 bits_device, g->row_begin,
                                                                                 g->row_begin + g->n_rows);
        CU(cudaGetLastError());
    }
    k_clear_remote_flags<<<grid_for(g->n_global, 256, num_sms() * 8), 256, 0, g->stream>>>(g->flags, g->n_global, g->row_begin,
                                                                                        g->row_begin + g->n_rows);
    CU(cudaGetLastError());
    return NULPA_OK;
}

int nulpa_or_flag_bits(nulpa_graph *g, const uint32_t *bits_device, int P, int64_t words) {
    if (!g || !bits_device || P < 1 || words * 32 < g->n_rows) return fail(NULPA_EINVAL, "bad argument");
    if (g->n_rows > 0) {
        k_or_flag_bits<<<grid_for(g->n_rows, 256, num_sms() * 8), 256, 0, g->stream>>>(g->flags, bits_device, P, words,
                                                                                     g->row_begin, g->row_begin + g->n_rows);
        CU(cudaGetLastError());
    }
    return NULPA_OK;
}

int nulpa_bind_state(nulpa_graph *g, int32_t *labels_device, uint8_t *flags_device) {
    if (!g || !labels_device || !flags_device) return fail(NULPA_EINVAL, "null argument");
    g->labels = labels_device;
    g->flags = flags_device;
    return NULPA_OK;
}

int nulpa_reset(nulpa_graph *g) {
    if (!g) return fail(NULPA_EINVAL, "null handle");
    return reset_state(g);
}

int nulpa_sweep(nulpa_graph *g, int pickless, const nulpa_params *params, int64_t *changed) {
    if (!g) return fail(NULPA_EINVAL, "null handle");
    nulpa_params p;
    if (params) p = *params; else nulpa_default_params(&p);
    CHECK(validate_params(p));
    CHECK(ensure_bins(g, p));
    unsigned long long *ctr = g->ctr + (size_t)kMaxIter * kCtr;   // spare slot
    CU(cudaMemsetAsync(ctr, 0, kCtr * sizeof(unsigned long long), g->stream));
    CHECK(sweep(g, pickless ? 1 : 0, p, ctr, false, 0));
    if (changed) {
        CU(cudaMemcpyAsync(g->ctr_host, ctr, kCtr * sizeof(unsigned long long), cudaMemcpyDeviceToHost, g->stream));
        CU(cudaStreamSynchronize(g->stream));
        *changed = (int64_t)g->ctr_host[0];
        for (int b = 0; b < 4; ++b) {
            g->stats.vertices_processed[b] += (int64_t)g->ctr_host[1 + b];
            g->stats.edges_scanned[b] += (int64_t)g->ctr_host[5 + b];
            g->stats.vertices_changed[b] += (int64_t)g->ctr_host[9 + b];
            g->stats.changed_edges[b] += (int64_t)g->ctr_host[13 + b];
        }
    }
    return NULPA_OK;
}

int nulpa_run(nulpa_graph *g, const nulpa_params *params, nulpa_stats *stats) {
    if (!g) return fail(NULPA_EINVAL, "null handle");
    nulpa_params p;
    if (params) p = *params; else nulpa_default_params(&p);
    CHECK(validate_params(p));
    CHECK(ensure_bins(g, p));
    const int maxit = std::min(p.max_iterations, kMaxIter);
    if (p.max_iterations > kMaxIter) return fail(NULPA_EINVAL, "max_iterations must be <= %d", kMaxIter);
    zero_stats_counts(&g->stats);
    CHECK(ensure_events(g));
    const bool timing = p.timing != 0;
    CU(cudaMemsetAsync(g->ctr, 0, (size_t)(kMaxIter + 1) * kCtr * sizeof(unsigned long long), g->stream));
    CU(cudaEventRecord(g->ev_run[0], g->stream));
    if (p.reset) CHECK(reset_state(g));
    int l = 0;
    int converged = 0;
    // the device loop's CUDA graph is captured and instantiated once per
    // handle and parameter set (~tens of ms): a handle's first run takes the
    // host loop, so a one-shot create -> run -> destroy (the end-to-end path)
    // does not pay for a graph it uses once; later runs build and replay it
    const bool dloop = !timing && p.device_loop && maxit >= 2 &&
                       (g->runs > 0 || (g->loop_exec && same_loop_params(g->loop_p, p) && g->loop_p.max_iterations == maxit));
    ++g->runs;
    if (dloop) {
        // device loop: sweep 0 (first-sweep schedule) from the host, then
        // one graph launch runs the stop tests and sweeps 1.. (no host sync
        // per iteration)
        const int pl0 = p.pickless_period > 0;
        unsigned long long *scratch = g->ctr + (size_t)kMaxIter * kCtr;
        if (!g->loopvars) CHECK(dalloc(&g->loopvars, 4));
        CU(cudaMemsetAsync(g->loopvars, 0, 4 * sizeof(int32_t), g->stream));
        if (pl0) CU(cudaMemsetAsync(g->loopvars + 1, 1, 1, g->stream));   // lv[1] = 1 (little-endian)
        CHECK(sweep(g, pl0, p, scratch, false, 0));
        if (!g->loop_exec || !same_loop_params(g->loop_p, p) || g->loop_p.max_iterations != maxit)
            CHECK(build_loop(g, p, maxit));
        CU(cudaGraphLaunch(g->loop_exec, g->stream));
        int32_t lv[4];
        CU(cudaMemcpyAsync(lv, g->loopvars, sizeof lv, cudaMemcpyDeviceToHost, g->stream));
        CU(cudaStreamSynchronize(g->stream));
        l = lv[3];
        converged = lv[2];
        for (int b = 0; b < 4; ++b) g->stats.launches[b] += g->loop_launches[b] * (l - 1);
        g->stats.other_launches += g->loop_other * (l - 1) + 1;
        g->sweeps_since_reset += l - 1;
    }
    for (; l < maxit && !dloop; ++l) {
        const int pl = p.pickless_period > 0 && (l % p.pickless_period) == 0;
        unsigned long long *ctr = g->ctr + (size_t)l * kCtr;
        CHECK(sweep(g, pl, p, ctr, timing, l));
        CU(cudaMemcpyAsync(g->ctr_host + (size_t)l * kCtr, ctr, sizeof(unsigned long long), cudaMemcpyDeviceToHost, g->stream));
        CU(cudaStreamSynchronize(g->stream));
        const int64_t dn = (int64_t)g->ctr_host[(size_t)l * kCtr];
        if (!pl && (double)dn / (double)g->n_global < p.tolerance) {
            ++l;
            converged = 1;
            break;
        }
    }
    CU(cudaEventRecord(g->ev_run[1], g->stream));
    CU(cudaMemcpyAsync(g->ctr_host, g->ctr, (size_t)kMaxIter * kCtr * sizeof(unsigned long long), cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    nulpa_stats &s = g->stats;
    s.iterations = l;
    s.converged = converged;
    for (int it = 0; it < l; ++it) {
        const unsigned long long *c = g->ctr_host + (size_t)it * kCtr;
        s.changed[it] = (int64_t)c[0];
        for (int b = 0; b < 4; ++b) {
            s.vertices_processed[b] += (int64_t)c[1 + b];
            s.edges_scanned[b] += (int64_t)c[5 + b];
            s.vertices_changed[b] += (int64_t)c[9 + b];
            s.changed_edges[b] += (int64_t)c[13 + b];
            s.iter_processed[it][b] = (int64_t)c[1 + b];
            s.iter_edges[it][b] = (int64_t)c[5 + b];
            s.iter_changed[it][b] = (int64_t)c[9 + b];
            s.iter_changed_edges[it][b] = (int64_t)c[13 + b];
        }
        if (timing) {
            for (int b = 0; b < 4; ++b) {
                float ms = 0;
                CU(cudaEventElapsedTime(&ms, g->ev[(it * 4 + b) * 2], g->ev[(it * 4 + b) * 2 + 1]));
                s.kernel_ms[b] += ms;
                s.iter_kernel_ms[it][b] = ms;
            }
        }
    }
    float rms = 0;
    CU(cudaEventElapsedTime(&rms, g->ev_run[0], g->ev_run[1]));
    s.run_ms = rms;
    if (stats) *stats = s;
    return NULPA_OK;
}

int nulpa_labels(nulpa_graph *g, int32_t *out, int memkind) {
    if (!g || !out) return fail(NULPA_EINVAL, "null argument");
    CHECK(resolve_mem(out, memkind));
    CU(cudaMemcpyAsync(out, g->labels, g->n_global * sizeof(int32_t),
                       memkind == NULPA_MEM_HOST ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    return NULPA_OK;
}

int nulpa_flags(nulpa_graph *g, uint8_t *out, int memkind) {
    if (!g || !out) return fail(NULPA_EINVAL, "null argument");
    CHECK(resolve_mem(out, memkind));
    CU(cudaMemcpyAsync(out, g->flags, g->n_global,
                       memkind == NULPA_MEM_HOST ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    return NULPA_OK;
}

int nulpa_set_labels(nulpa_graph *g, const int32_t *in, const uint8_t *flags, int memkind) {
    if (!g || !in) return fail(NULPA_EINVAL, "null argument");
    CHECK(resolve_mem(in, memkind));
    CHECK(check_labels(g, in, memkind));
    const cudaMemcpyKind k = memkind == NULPA_MEM_HOST ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
    CU(cudaMemcpyAsync(g->labels, in, g->n_global * sizeof(int32_t), k, g->stream));
    if (flags)
        CU(cudaMemcpyAsync(g->flags, flags, g->n_global, k, g->stream));
    else
        CU(cudaMemsetAsync(g->flags, 1, g->n_global, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    return NULPA_OK;
}

}  // extern "C"

namespace {
int modularity_partial(nulpa_graph *g, const int32_t *lab, double *sigma_intra, double *two_m, double *Sigma_device) {
    if (!g->macc) CHECK(dalloc(&g->macc, 4));
    CU(cudaMemsetAsync(g->macc, 0, 4 * sizeof(double), g->stream));
    const int sms = num_sms();
    if (!g->Kdeg) {                                         // graph-invariant: K_i and 2m, once
        CHECK(dalloc(&g->Kdeg, (size_t)std::max<int64_t>(g->n_rows, 1)));
        if (g->weights)
            k_mod_degrees<true><<<sms * 8, 256, 0, g->stream>>>(g->offsets, g->weights, g->n_rows, g->Kdeg, g->macc);
        else
            k_mod_degrees<false><<<sms * 8, 256, 0, g->stream>>>(g->offsets, g->weights, g->n_rows, g->Kdeg, g->macc);
        CU(cudaGetLastError());
        double h2[4];
        CU(cudaMemcpyAsync(h2, g->macc, sizeof h2, cudaMemcpyDeviceToHost, g->stream));
        CU(cudaStreamSynchronize(g->stream));
        g->two_m_local = h2[1];
        CU(cudaMemsetAsync(g->macc, 0, 4 * sizeof(double), g->stream));
    }
    if (g->weights)
        k_mod_intra<true><<<sms * 8, 256, 0, g->stream>>>(g->offsets, g->indices, g->weights, lab, g->n_rows, g->row_begin, g->macc);
    else
        k_mod_intra<false><<<sms * 8, 256, 0, g->stream>>>(g->offsets, g->indices, g->weights, lab, g->n_rows, g->row_begin, g->macc);
    k_mod_sigma<<<sms * 8, 256, 0, g->stream>>>(g->Kdeg, lab, g->n_rows, g->row_begin, Sigma_device);
    CU(cudaGetLastError());
    double h[4];
    CU(cudaMemcpyAsync(h, g->macc, sizeof h, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    *sigma_intra += h[0];
    *two_m += g->two_m_local;
    return NULPA_OK;
}
}  // namespace

extern "C" {

int nulpa_modularity_partial(nulpa_graph *g, const int32_t *labels_device, double *sigma_intra, double *two_m,
                             double *Sigma_device) {
    if (!g || !sigma_intra || !two_m || !Sigma_device) return fail(NULPA_EINVAL, "null argument");
    if (labels_device) CHECK(check_labels(g, labels_device, NULPA_MEM_DEVICE));
    return modularity_partial(g, labels_device ? labels_device : g->labels, sigma_intra, two_m, Sigma_device);
}

int nulpa_modularity_finish(nulpa_graph *g, const double *Sigma_device, double sigma_intra, double two_m, double *q) {
    if (!g || !Sigma_device || !q) return fail(NULPA_EINVAL, "null argument");
    if (!g->macc) CHECK(dalloc(&g->macc, 4));
    CU(cudaMemsetAsync(g->macc, 0, 4 * sizeof(double), g->stream));
    k_mod_finish<<<grid_for(g->n_global, 256, num_sms() * 8), 256, 0, g->stream>>>(const_cast<double *>(Sigma_device), g->n_global, g->macc, 0);
    CU(cudaGetLastError());
    double h[4];
    CU(cudaMemcpyAsync(h, g->macc, sizeof h, cudaMemcpyDeviceToHost, g->stream));
    CU(cudaStreamSynchronize(g->stream));
    *q = two_m > 0 ? sigma_intra / two_m - h[2] / (two_m * two_m) : 0.0;
    return NULPA_OK;
}

int nulpa_modularity(nulpa_graph *g, const int32_t *labels, int memkind, double *q) {
    if (!g || !q) return fail(NULPA_EINVAL, "null argument");
    if (g->n_rows != g->n_global) return fail(NULPA_ESTATE, "nulpa_modularity needs a whole graph; use the _partial/_finish pair for shards");
    const int32_t *lab = g->labels;
    int32_t *tmp = nullptr;
    if (labels) {
        CHECK(resolve_mem(labels, memkind));
        CHECK(check_labels(g, labels, memkind));
        if (memkind == NULPA_MEM_HOST) {
            CHECK(dalloc(&tmp, (size_t)g->n_global));
            CU(cudaMemcpyAsync(tmp, labels, g->n_global * sizeof(int32_t), cudaMemcpyHostToDevice, g->stream));
            lab = tmp;
        } else {
            lab = labels;
        }
    }
    if (!g->Sigma) CHECK(dalloc(&g->Sigma, (size_t)g->n_global));
    if (!g->macc) CHECK(dalloc(&g->macc, 4));
    CU(cudaMemsetAsync(g->Sigma, 0, g->n_global * sizeof(double), g->stream));
    double sigma = 0, two_m = 0;
    int r = modularity_partial(g, lab, &sigma, &two_m, g->Sigma);
    if (r == NULPA_OK) r = nulpa_modularity_finish(g, g->Sigma, sigma, two_m, q);
    dfree(tmp);
    return r;
}

int nulpa_release_memory(void) {
    cudaMemPool_t pool = device_pool();
    if (pool) CU(cudaMemPoolTrimTo(pool, 0));
    return NULPA_OK;
}

int nulpa_get_stats(nulpa_graph *g, nulpa_stats *out) {
    if (!g || !out) return fail(NULPA_EINVAL, "null argument");
    *out = g->stats;
    return NULPA_OK;
}

int nulpa_state_pointers(nulpa_graph *g, int32_t **labels_device, uint8_t **flags_device) {
    if (!g) return fail(NULPA_EINVAL, "null handle");
    if (labels_device) *labels_device = g->labels;
    if (flags_device) *flags_device = g->flags;
    return NULPA_OK;
}

int nulpa_destroy(nulpa_graph *g) {
    if (!g) return NULPA_OK;
    if (g->stream) cudaStreamSynchronize(g->stream);
    free_bins(g);
    dfree(g->loopvars);
    if (g->cap) {
        cudaStreamSynchronize(g->cap);
        cudaStreamDestroy(g->cap);
    }
    if (g->own_csr) {
        dfree(g->offsets);
        dfree(g->indices);
        dfree(g->weights);
    }
    dfree(g->own_labels);
    dfree(g->own_flags);
    dfree(g->labels_prev);
    dfree(g->flags_prev);
    dfree(g->ctr);
    if (g->ctr_host) cudaFreeHost(g->ctr_host);
    dfree(g->Sigma);
    dfree(g->macc);
    dfree(g->Kdeg);
    if (g->hi) {
        cudaStreamSynchronize(g->hi);
        cudaStreamDestroy(g->hi);
        cudaEventDestroy(g->ev_mid);
        cudaEventDestroy(g->ev_join2);
    }
    if (g->side) {
        cudaStreamSynchronize(g->side);
        cudaStreamDestroy(g->side);
        cudaEventDestroy(g->ev_fork);
        cudaEventDestroy(g->ev_join);
    }
    if (g->events) {
        for (auto &e : g->ev) cudaEventDestroy(e);
        cudaEventDestroy(g->ev_run[0]);
        cudaEventDestroy(g->ev_run[1]);
    }
    delete g;
    return NULPA_OK;
}

}  // extern "C"
