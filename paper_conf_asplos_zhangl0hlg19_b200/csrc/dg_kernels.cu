// DiGraph hot path on sm_100a (B200): the persistent path-propagation kernel
// with device-side activity tracking and convergence counter, the
// vertex-centric ablation, and the multi-GPU boundary pack/unpack kernels.
//
// Path-based asynchronous execution (sec. 3.1, lines 94-96): the
// vertices of a path are handled in path order inside one round, so a new
// state reaches the path's later vertices in the same round.  B200 mapping
// (DESIGN.md "Kernels"): one warp walks a partition (a run of whole paths,
// "the threads of a warp (assigned with a partition) read
// consecutive data") in windows of 128 path entries; lane l owns entries
// 4l..4l+3 (16-byte vector loads of e_idx / e_w / S_val), gathers their master
// states, and the in-order walk along every path is computed exactly as a
// segmented warp scan (shuffles) of per-entry transfer functions:
//   SSSP/BFS/WCC/SCC  x_i = min(a_i, x_(i-1) + w_i)      (min-plus, heads reset)
//   PR/Adsorption     a_i = alpha_i + beta_i * a_(i-1)   (affine, heads reset)
// Masters (V_val) change only through atomicMin/atomicAdd.
// A master whose state changed sets its bit in the next round's signal
// bitmap; a window is walked in a round only if one of its vertices was
// signalled (or a path carries a live value into it), so converged regions
// cost one streamed 4-byte index per entry.  All rounds run inside one
// cooperative persistent launch; partitions are dispatched from a device
// ticket in priority order (layer, then hotness: PAPER.md lines 169, 192) and
// the run ends when a round signals no vertex (device-side active counter,
// north_star (4)).
#include <cooperative_groups.h>
#include <cub/device/device_scan.cuh>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <tuple>

#include "dg_internal.h"

namespace cg = cooperative_groups;

namespace dg {

#define CK(call)                                                                              \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess) {                                                              \
            err = std::string(#call) + ": " + cudaGetErrorString(e_);                         \
            return DG_ENOCUDA;                                                                \
        }                                                                                     \
    } while (0)

constexpr uint32_t INF = DG_INF;
constexpr int kBlock = 256;
constexpr int kWarps = kBlock / 32;
constexpr int kPad = 256;  // zero entries after every per-entry array
#ifndef DG_PATH_MINB
#define DG_PATH_MINB 3  // resident CTAs per SM requested for the path kernel
#endif

// device counters of a run
struct Counters {
    unsigned long long updates, edges, units, entries, pushes;
    unsigned int active[2];  // path mode: non-zero iff bitmap[k] has a signalled vertex (an upper bound on
                             // their number: a vertex lowered twice counts twice); vertex mode: frontier sizes
    unsigned int ticket[2];
    unsigned int minval[2];  // SSSP/BFS: smallest distance signalled into bitmap[k] (bucket base of its round)
    unsigned int qn[2];      // SSSP/BFS sparse rounds: length of the round's compacted frontier list
    unsigned int osum[2];    // ... and the occurrences (out-edges) of its vertices
    unsigned int qcur[2];    // append cursor of the list
    unsigned int qn_in[2], osum_in[2], qcur_in[2], ticket_in[2];  // WCC sparse rounds: the in-edge phase
    int round;  // global round number of the next round
    int pad;
    // fused multi-rank runs (path_kernel with P.mr.world > 1)
    unsigned long long mr_dirty;  // boundary values changed since the last exchange (this rank)
    unsigned long long mr_total;  // all ranks' published activity at the last exchange
    unsigned long long mr_ex;     // exchanges done by the last launch
    unsigned long long mr_err;    // a peer did not arrive (timeout)
    unsigned long long dense_rounds;  // rounds that streamed every window's path entries (not sparse)
};

struct DevWork {
    uint32_t* vs_u = nullptr;              // SSSP/BFS dist, WCC/SCC label (4 B: twice the masters per L2 sector)
    uint32_t* vstamp = nullptr;            // vertex-centric ablation: round a vertex was last queued
    float4* vs_f = nullptr;                // vertex-centric ablation: {r, g, delta, stamp}
    unsigned long long* vs_t = nullptr;    // path-mode PR / Adsorption masters: exact fixed-point totals T
    unsigned long long* sigma = nullptr;   // T at the vertex's last signal
    unsigned long long* s_val = nullptr;   // per-entry mirrors S_val (Fig. 4)
    unsigned long long* bnd_base = nullptr;
    float* e_coef = nullptr;               // Adsorption: coefficient of the path edge out of each entry
    float* pr_coef = nullptr;              // PageRank: d/outdeg(v_i) of the path edge out of each entry
    double pr_coef_d = -1.0;               // the damping pr_coef was computed for
    float* ads_base = nullptr;             // Adsorption: p_inj * I
    uint32_t* bits = nullptr;              // 2 x nw signal bitmaps
    int64_t nw = 0;
    int32_t* vlist[2] = {nullptr, nullptr};  // ablation frontiers
    Counters* ctr = nullptr;
    Counters* ctr_host = nullptr;          // mapped pinned mirror the path kernel writes at its end
    Counters* ctr_host_dev = nullptr;      // ... its device address
    bool ctr_mirror_fresh = false;         // the mirror holds the counters of the last path launch
    bool defer_kernel_time = false;        // coop_launch leaves the kernel events to the caller (dg_run)
    bool kernel_time_pending = false;
    double* dsum = nullptr;
    int32_t* scc_label = nullptr;
    uint8_t* scc_mark = nullptr;
    int32_t* remaining = nullptr;
    uint32_t* out_stage = nullptr;         // dg_get_states staging buffer (n words)
    void* host_stage = nullptr;            // dg_get_states pinned host staging (n words)
    int64_t host_stage_n = 0;
    unsigned* qtick = nullptr;             // per-CTA partition queue counters (2 x kMaxGrid x kQStride)
    uint32_t* occ_off = nullptr;           // vertex -> its non-tail path entries (sparse rounds), n+1
    uint32_t* occ = nullptr;               // entry indices grouped by vertex
    uint2* occ_items = nullptr;            // frontier items (v, chunk of <= kOccChunk occurrences)
    uint2* e_cw = nullptr;                 // SSSP sparse rounds: {e_idx, e_w} interleaved (one load per step)
    bool cw_ok = false;
    uint32_t* iocc_off = nullptr;          // vertex -> its non-head path entries (SCC backward), n+1
    uint32_t* iocc = nullptr;
    bool iocc_ok = false;
    int64_t occ_cap = 0, iocc_cap = 0;     // allocated lengths of occ / iocc
    uint32_t* occ_cur = nullptr;           // index build scratch
    void* cub_tmp = nullptr;
    size_t cub_tmp_bytes = 0;
    bool occ_ok = false;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr, kev0 = nullptr, kev1 = nullptr;
    bool have_params = false;
};

// Peer-memory exchange region (see "peer-memory boundary exchange" below):
// header (u64 words): [0, kP2PMaxRanks) epochs written by the peers, [16]
// error word, [17 + parity] this rank's published activity; then two slots.
constexpr int kP2PMaxRanks = 16;
constexpr size_t kP2PHeader = 256;
constexpr int kP2PErr = kP2PMaxRanks, kP2PCount = kP2PMaxRanks + 1;
// Fused multi-rank run: the exchange happens inside path_kernel's round loop.
struct MultiRank {
    const unsigned char* region[kP2PMaxRanks];  // every rank's region in this address space (own included)
    unsigned long long* own;                    // this rank's region
    const int32_t* bnd;                         // boundary vertices (internal ids), identical on every rank
    const unsigned long long* hold;             // holder ranks of each boundary vertex (bit r: rank r)
    unsigned long long* base;                   // SUM: total after the last exchange
    uint32_t* last;                             // MIN: reduced value of the last exchange
    int64_t nb;
    unsigned long long slot_bytes, epoch0, timeout_ns, eps_fx;
    int world, rank, every, sum;
    int mark;  // SCC backward phase: the replicated state is the reachability mark (value 0 = marked, MIN = OR)
};

struct KParams {
    const uint32_t* e_idx;
    const int32_t* e_w;
    const int64_t* part_off;
    const int64_t* row_ptr;
    const int32_t* col;
    const int32_t* w;
    int64_t n_part, n, nw;
    uint32_t* vs_u;
    uint32_t* vstamp;
    float4* vs_f;
    unsigned long long* vs_t;
    unsigned long long* sigma;
    unsigned long long* s_val;
    const float* e_coef;
    uint32_t* bits;  // bits[0..nw) and bits[nw..2nw)
    int32_t* vlist0;
    int32_t* vlist1;
    Counters* ctr;
    uint8_t* mark;
    const int32_t* scc_label;
    const int32_t* orig;
    int64_t n_proxy;
    float eps;
    unsigned long long eps_fx;
    int max_rounds;
    int px_refresh;  // partitions a CTA walks between mid-round proxy flushes (0: round end only)
    int part_order;  // 0: priority order; 1: reversed; k > 1: t -> t*k mod n_part (k coprime to n_part)
    uint64_t hot_master_bytes;  // evict-last prefix of the accumulative masters
    uint32_t delta;  // SSSP/BFS bucket width (reading R-DELTA); 0 = unbounded
    const uint32_t* occ_off;  // SSSP/BFS sparse rounds: occurrence index (null: dense rounds only)
    const uint32_t* occ;
    uint2* occ_items;         // the round's frontier items (v, chunk)
    const uint2* e_cw;        // SSSP sparse walk: path entry code and weight in one 8-byte word (null: separate)
    const uint32_t* iocc_off;  // WCC: the in-edge occurrence index as well
    const uint32_t* iocc;
    uint32_t sparse_max;      // rounds with at most this many signalled vertices are candidates (n/4)
    uint32_t sparse_occ;      // ... and are walked sparse if their out-edges are at most this many
    int sparse_walk;          // path edges a sparse walk follows at most
    uint32_t probe_free_occ;  // min-plus dense rounds whose signalled vertices own at least this many
                              // out-edges (or that signal more than sparse_max vertices) walk every
                              // window without probing the bitmap (0: always probe)
    uint32_t probe_free_act;  // ... or that signalled more than this many vertices (n/4)
    MultiRank mr;             // world > 1: fused multi-rank run
    unsigned* qtick;            // per-CTA partition queue counters, 2 x grid x kQStride (null: global ticket)
    unsigned long long* trace;  // DG_TRACE: per round {end time ns, vertices signalled into it, dense, out-edges}
    int trace_cap;
    unsigned long long* snap;  // DG_EXP 32/64: master snapshots gathered instead of the live masters (2 x n)
    Counters* ctr_out;  // mapped host mirror of *ctr written at the end of the launch (null: none)
    int exp;  // -DDG_EXP builds only (scripts/build_exp.sh): cost-breakdown switches, DG_EXP bitmask
};
__device__ int g_exp_par;  // DG_EXP 32/64: the snapshot buffer gathered this round
#ifdef DG_EXP
#define EXP_ON(P, b) (((P).exp & (b)) != 0)
#else
#define EXP_ON(P, b) false
#endif

// ------------------------------------------------------------------ helpers
__device__ __forceinline__ uint32_t sat_add(uint32_t a, uint32_t b) {
    uint32_t s = a + b;  // a, b <= INF = 2^31-1: no wrap
    return s < INF ? s : INF;
}
__device__ __forceinline__ uint4 ld_stream_u4(const uint32_t* p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ int4 ld_stream_i4(const int32_t* p) {
    int4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ float4 ld_stream_f4(const float* p) {
    float4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
    return r;
}
__device__ __forceinline__ void ld_stream_u64x4(const unsigned long long* p, unsigned long long (&o)[4]) {
    asm volatile("ld.global.L1::no_allocate.v2.u64 {%0,%1}, [%2];" : "=l"(o[0]), "=l"(o[1]) : "l"(p));
    asm volatile("ld.global.L1::no_allocate.v2.u64 {%0,%1}, [%2];" : "=l"(o[2]), "=l"(o[3]) : "l"(p + 2));
}
// L2 eviction policies: streamed path arrays are evict-first so they do not
// push the (re-used) vertex states out of the 126 MB L2; states are evict-last.
__device__ __forceinline__ unsigned long long policy_evict_first() {
    unsigned long long p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ unsigned long long policy_evict_last() {
    unsigned long long p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// Masters: evict-last for the hot prefix of the degree-ordered state array
// (the vertices most entries touch), unchanged priority for the cold tail --
// when the states exceed L2 (Twitter scale) the hot prefix stays resident.
__device__ __forceinline__ unsigned long long policy_masters(const void* base, uint32_t hot_bytes, uint32_t total) {
    unsigned long long p;
    asm volatile("createpolicy.range.global.L2::evict_last.L2::evict_unchanged.b64 %0, [%1], %2, %3;"
                 : "=l"(p) : "l"(base), "r"(hot_bytes), "r"(total));
    return p;
}
__device__ __forceinline__ void red_add_u64_h(unsigned long long* p, unsigned long long v, unsigned long long pol) {
    asm volatile("red.global.add.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(p), "l"(v), "l"(pol) : "memory");
}
__device__ __forceinline__ uint4 ld_stream_u4_h(const uint32_t* p, unsigned long long pol) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
    return r;
}
__device__ __forceinline__ float4 ld_stream_f4_h(const float* p, unsigned long long pol) {
    float4 r;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p), "l"(pol));
    return r;
}
// 256-bit (sm_100) vector load/store of a lane's four 64-bit mirrors
__device__ __forceinline__ void ld_stream_u64x4_h(const unsigned long long* p, unsigned long long (&o)[4],
                                                  unsigned long long pol) {
    asm volatile("ld.global.L1::no_allocate.L2::cache_hint.v4.u64 {%0,%1,%2,%3}, [%4], %5;"
                 : "=l"(o[0]), "=l"(o[1]), "=l"(o[2]), "=l"(o[3]) : "l"(p), "l"(pol));
}
__device__ __forceinline__ void st_stream_u64x4_h(unsigned long long* p, const unsigned long long (&v)[4],
                                                  unsigned long long pol) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.v4.u64 [%0], {%1,%2,%3,%4}, %5;"
                 ::"l"(p), "l"(v[0]), "l"(v[1]), "l"(v[2]), "l"(v[3]), "l"(pol));
}
__device__ __forceinline__ void st_stream_u64_h(unsigned long long* p, unsigned long long v, unsigned long long pol) {
    asm volatile("st.global.L1::no_allocate.L2::cache_hint.u64 [%0], %1, %2;" ::"l"(p), "l"(v), "l"(pol));
}
__device__ __forceinline__ uint32_t u4get(const uint4& v, int k) {
    return k == 0 ? v.x : k == 1 ? v.y : k == 2 ? v.z : v.w;
}
__device__ __forceinline__ int32_t i4get(const int4& v, int k) {
    return k == 0 ? v.x : k == 1 ? v.y : k == 2 ? v.z : v.w;
}
__device__ __forceinline__ float f4get(const float4& v, int k) {
    return k == 0 ? v.x : k == 1 ? v.y : k == 2 ? v.z : v.w;
}
__device__ __forceinline__ bool test_bit(const uint32_t* b, uint32_t v) { return (b[v >> 5] >> (v & 31)) & 1u; }
// set v's bit in the next round's bitmap; true if this call set it
__device__ __forceinline__ bool signal_vertex(uint32_t* b, uint32_t v) {
    const uint32_t m = 1u << (v & 31);
    return !(atomicOr(&b[v >> 5], m) & m);
}

// per-thread statistics (32-bit: a thread's share stays far below 2^32;
// widened to 64 bits for the warp reduction)
struct Acc {
    unsigned upd = 0, edges = 0, units = 0, entries = 0, pushes = 0;
    unsigned sig = 0;
    uint32_t vmin = 0x7FFFFFFFu;  // SSSP/BFS: smallest distance committed this round
};

// ------------------------------------------------------------------ path walks
// cp.async (sm_80+ LDGSTS): 16-byte global -> shared copies that hold no
// registers while in flight; L2-only (.cg), with an L2 eviction policy.
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, unsigned long long pol) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(s), "l"(gmem), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// Partition dispatch of a dense round ("work stealing
// for balanced load between SMXs", line 192 priority order; north_star (3)
// "per-SM hot-first priority work queue").  The partitions are in priority
// order; CTA c owns the queue {c, c+G, c+2G, ...} (G = grid size), so every
// queue is itself hot-first and all CTAs advance through the priority order
// together.  A CTA's warps take partitions from its own queue (one atomic on
// the CTA's own counter, on its own 32-byte line); once it is empty they steal
// single partitions from the other CTAs' queues, starting at the next CTA, and
// a per-CTA shared cursor skips victims found empty.  This is DG_DISPATCH=1
// (developer knob); the default is one global ticket, which measured faster
// (the accumulative walk also prefetches its tickets a partition ahead).
struct Queue {
    unsigned* qt;        // per-CTA counters of this round (stride kQStride)
    unsigned* global;    // the single global ticket (DG_DISPATCH=0)
    unsigned* s_state;   // shared: [0] next victim offset, [1] own queue empty
};
constexpr int kQStride = 8;
constexpr int kMaxGrid = 4096;  // CTAs of a persistent launch (148 SMs x resident CTAs)
constexpr unsigned kNoPart = 0xFFFFFFFFu;
__device__ __forceinline__ unsigned queue_len(unsigned n_part, unsigned c, unsigned G) {
    return n_part > c ? (n_part - c - 1) / G + 1 : 0u;
}
// The rank (in priority order) of the warp's next partition, or kNoPart; all
// lanes call it.  Own queue: one atomic by lane 0.  Stealing: the warp probes
// 32 victims' counters at once with plain loads, then takes from the first
// with partitions left (atomic); a batch found empty advances the CTA's shared
// cursor, so each CTA scans the other queues about once per round.
__device__ __forceinline__ unsigned take_rank(const KParams& P, const Queue& q) {
    const unsigned np = (unsigned)P.n_part;
    const int lane = threadIdx.x & 31;
    unsigned t = kNoPart;
    if (!q.qt) {
        if (lane == 0) {
            const unsigned k = atomicAdd(q.global, 1u);
            t = k < np ? k : kNoPart;
        }
        return __shfl_sync(0xffffffffu, t, 0);
    }
    const unsigned G = gridDim.x, c = blockIdx.x;
    if (lane == 0 && !*(volatile unsigned*)&q.s_state[1]) {
        const unsigned k = atomicAdd(&q.qt[c * kQStride], 1u);
        if (k < queue_len(np, c, G)) t = c + k * G;
        else q.s_state[1] = 1u;
    }
    t = __shfl_sync(0xffffffffu, t, 0);
    if (t != kNoPart) return t;
    while (true) {
        const unsigned j0 = *(volatile unsigned*)&q.s_state[0];
        if (j0 >= G) return kNoPart;
        const unsigned j = j0 + lane;
        const unsigned v = c + j < G ? c + j : c + j - G;
        const bool left = j < G && __ldcg(&q.qt[v * kQStride]) < queue_len(np, v, G);
        unsigned mask = __ballot_sync(0xffffffffu, left);
        while (mask) {
            const int l = __ffs(mask) - 1;
            mask &= mask - 1;
            const unsigned vv = __shfl_sync(0xffffffffu, v, l);
            unsigned k = 0;
            if (lane == 0) k = atomicAdd(&q.qt[vv * kQStride], 1u);
            k = __shfl_sync(0xffffffffu, k, 0);
            if (k < queue_len(np, vv, G)) return vv + k * G;
        }
        if (lane == 0) atomicMax(&q.s_state[0], j0 + 32);
        __syncwarp();
    }
}
__device__ __forceinline__ unsigned next_partition(const KParams& P, const Queue& q) {
    unsigned t = take_rank(P, q);
    if (t == kNoPart) return kNoPart;
    if (P.part_order == 1) t = (unsigned)P.n_part - 1 - t;  // developer knob: dispatch-order experiments
    else if (P.part_order > 1) t = (unsigned)(((unsigned long long)t * P.part_order) % (unsigned long long)P.n_part);
    return t;
}

// A warp's stream of 128-entry windows over the partitions it takes from its
// queue: base == kNoWin marks the end of the stream.  Entry offsets are 32-bit
// (dev_upload_layout checks M + padding < 2^32) so the three cursors of the
// software pipeline stay in 9 registers.
constexpr uint32_t kNoWin = 0xFFFFFFFFu;
struct Win {
    uint32_t base, beg, end;
};
__device__ __forceinline__ Win win_first_of(const KParams& P, const Queue& q) {
    const unsigned t = next_partition(P, q);
    if (t == kNoPart) return Win{kNoWin, 0, 0};
    const uint32_t beg = (uint32_t)P.part_off[t], end = (uint32_t)P.part_off[t + 1];
    return Win{beg & ~3u, beg, end};
}
__device__ __forceinline__ Win win_next(const KParams& P, const Win& w, const Queue& q) {
    if (w.base == kNoWin) return w;
    if (w.base + 128 < w.end) return Win{w.base + 128, w.beg, w.end};
    return win_first_of(P, q);
}

// A warp's partition feed (both dense walks): with the global ticket
// (default) the ticket of the partition after next and the bounds of the next
// partition are fetched one partition early, so a partition switch waits for
// no atomic or load.  With per-CTA queues (DG_DISPATCH=1) the switch takes
// the next partition synchronously.
// With the global ticket the first two partitions of every warp are static
// (warp g of Gw takes ranks g and g + Gw) and the ticket hands out ranks from
// 2 Gw on, so a round starts with two independent bound loads instead of two
// dependent atomic + load round trips per warp (the stall at the start of
// every round of a small graph, profiles/r02h_sssp_rmat16.md).
struct Feed {
    unsigned t_pend;     // lane 0: rank of the partition after next (a ticket + 2 Gw, or static)
    uint32_t nbeg, nend; // bounds of the next partition (nbeg == kNoWin: none)
};
__device__ __forceinline__ unsigned feed_warps() { return gridDim.x * (blockDim.x >> 5); }
__device__ __forceinline__ unsigned feed_warp() { return blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); }
__device__ __forceinline__ unsigned map_order(const KParams& P, unsigned t) {
    if (P.part_order == 1) return (unsigned)P.n_part - 1 - t;  // developer knob: dispatch-order experiments
    if (P.part_order > 1) return (unsigned)(((unsigned long long)t * P.part_order) % (unsigned long long)P.n_part);
    return t;
}
__device__ __forceinline__ void feed_fetch(const KParams& P, const Queue& q, Feed& f) {
    // the pending ticket becomes the next partition; a new ticket is taken
    const unsigned t = __shfl_sync(0xffffffffu, f.t_pend, 0);
    if (t < (unsigned)P.n_part) {
        const unsigned u = map_order(P, t);
        f.nbeg = (uint32_t)P.part_off[u];
        f.nend = (uint32_t)P.part_off[u + 1];
    } else {
        f.nbeg = kNoWin;
        f.nend = 0;
    }
    if ((threadIdx.x & 31) == 0) f.t_pend = 2u * feed_warps() + atomicAdd(q.global, 1u);
}
// The warp's first window of a round and the primed feed (global ticket), or
// the first window from its queue (per-CTA queues)
__device__ __forceinline__ Win feed_start(const KParams& P, const Queue& q, Feed& f) {
    if (q.qt) return win_first_of(P, q);
    const unsigned g = feed_warp(), t0 = g;
    Win w{kNoWin, 0, 0};
    if (t0 < (unsigned)P.n_part) {
        const unsigned u = map_order(P, t0);
        const uint32_t beg = (uint32_t)P.part_off[u], end = (uint32_t)P.part_off[u + 1];
        w = Win{beg & ~3u, beg, end};
    }
    f.t_pend = g + feed_warps();  // static second partition
    feed_fetch(P, q, f);          // its bounds in flight; the first ticket taken
    return w;
}
__device__ __forceinline__ Win feed_next(const KParams& P, const Queue& q, const Win& w, Feed& f) {
    if (w.base == kNoWin) return w;
    if (w.base + 128 < w.end) return Win{w.base + 128, w.beg, w.end};
    if (q.qt) return win_first_of(P, q);
    const Win nw = f.nbeg == kNoWin ? Win{kNoWin, 0, 0} : Win{f.nbeg & ~3u, f.nbeg, f.nend};
    if (nw.base != kNoWin) feed_fetch(P, q, f);
    return nw;
}

// Min-plus walk.  MODE 0 SSSP (weights), 1 BFS (unit weights), 2 WCC (weight 0,
// also backward along every path edge), 3 SCC forward colouring (weight 0,
// assigned vertices -- scc_label >= 0 -- break their paths).
// The warp walks its stream of windows with a one-window lookahead: while
// window w is walked, the signal bits of window w+1 are tested and, if one is
// set, its master states are already in flight (read slightly early -- the
// asynchronous semantics of any concurrent update; atomicMin stays the
// authority), as are the indices of window w+2.
template <int MODE>
__device__ void walk_minplus(const KParams& P, const Queue& ticket, const uint32_t* bcur, uint32_t* bnxt,
                             uint32_t theta, Acc& acc, bool all) {
    const int lane = threadIdx.x & 31;
    const uint4 kFill = make_uint4(kHead | kTail, kHead | kTail, kHead | kTail, kHead | kTail);
    auto load_code = [&](const Win& w) {
        uint4 c = kFill;
        if (w.base != kNoWin && w.base + 4 * lane < w.end) c = ld_stream_u4(P.e_idx + w.base + 4 * lane);
        return c;
    };
    // signal-bitmap words of a window's entries (issued two windows ahead)
    // (a round that signalled most vertices -- `all` -- treats every entry as
    // signalled: every window would be walked anyway, and the probes are one
    // random L2 access per entry; walking an unsignalled vertex's edges only
    // repeats relaxations that cannot improve)
    auto probe_words = [&](const Win& w, const uint4& code, uint4& words) {
        words = make_uint4(0u, 0u, 0u, 0u);
        if (w.base == kNoWin) return;
        if (all) {
            const uint32_t i = w.base + 4 * lane;
            words = make_uint4(i >= w.beg && i < w.end ? ~0u : 0u, i + 1 >= w.beg && i + 1 < w.end ? ~0u : 0u,
                               i + 2 >= w.beg && i + 2 < w.end ? ~0u : 0u, i + 3 >= w.beg && i + 3 < w.end ? ~0u : 0u);
            return;
        }
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t i = w.base + 4 * lane + k;
            const uint32_t wd = (i >= w.beg && i < w.end) ? bcur[(u4get(code, k) & kVMask) >> 5] : 0u;
            if (k == 0) words.x = wd; else if (k == 1) words.y = wd; else if (k == 2) words.z = wd; else words.w = wd;
        }
    };
    // the window's signal bits; if one is set, issue its master gathers (one window ahead)
    auto probe_finish = [&](const Win& w, const uint4& code, const uint4& words, bool (&act)[4], uint32_t (&a)[4]) {
        bool any = false;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t v = u4get(code, k) & kVMask;
            act[k] = (u4get(words, k) >> (v & 31)) & 1u;
            any |= act[k];
        }
        any = __any_sync(0xffffffffu, any);
        if (any) {
#pragma unroll
            for (int k = 0; k < 4; k++) {
                const uint32_t i = w.base + 4 * lane + k;
                a[k] = (i >= w.beg && i < w.end) ? P.vs_u[u4get(code, k) & kVMask] : INF;
            }
        }
        return any;
    };

    // pipeline: indices three windows ahead, bitmap words two ahead, masters one ahead
    Feed f{0u, kNoWin, 0u};
    Win wc = feed_start(P, ticket, f);
    if (wc.base == kNoWin) return;
    Win wn = feed_next(P, ticket, wc, f);
    Win wn2 = feed_next(P, ticket, wn, f);
    uint4 code_c = load_code(wc), code_n = load_code(wn), code_n2 = load_code(wn2);
    uint4 words_c, words_n;
    probe_words(wc, code_c, words_c);
    probe_words(wn, code_n, words_n);
    bool act_c[4], act_n[4];
    uint32_t a_c[4] = {INF, INF, INF, INF}, a_n[4] = {INF, INF, INF, INF};
    bool any_c = probe_finish(wc, code_c, words_c, act_c, a_c);
    uint32_t carry = INF, carry_vtx = 0;
    bool carry_live = false;
    while (wc.base != kNoWin) {
        const Win wn3 = feed_next(P, ticket, wn2, f);
        const uint4 code_n3 = load_code(wn3);
        uint4 words_n2;
        probe_words(wn2, code_n2, words_n2);
        const bool any_n = probe_finish(wn, code_n, words_n, act_n, a_n);
        if (wc.base == (wc.beg & ~3u)) { carry = INF; carry_live = false; }  // partition start
        const uint32_t i0 = wc.base + 4 * lane;
        // WCC looks one entry ahead: the path edge into the next window is walked backwards too
        uint32_t nx_lab = INF;
        bool nx_act = false;
        if (MODE == 2 && lane == 31) {
            const uint32_t inx = wc.base + 128;
            if (inx < wc.end) {
                const uint32_t nx_code = P.e_idx[inx];
                if (!(nx_code & kHead)) {
                    nx_act = test_bit(bcur, nx_code & kVMask);
                    nx_lab = P.vs_u[nx_code & kVMask];
                }
            }
        }
        const bool nx_any = MODE == 2 ? __any_sync(0xffffffffu, nx_act) : false;
        const bool walk = any_c || carry_live || nx_any;
        if (walk) {
            acc.units++;
            if (!any_c) {  // walked only for a live carry (or WCC look-ahead): gather now
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    const uint32_t i = i0 + k;
                    a_c[k] = (i >= wc.beg && i < wc.end) ? P.vs_u[u4get(code_c, k) & kVMask] : INF;
                }
            }
            int4 wv = make_int4(0, 0, 0, 0);
            if (MODE == 0 && i0 < wc.end) wv = ld_stream_i4(P.e_w + i0);
            uint32_t vtx[4], a[4], wgt[4];
            bool hd[4], tl[4], live[4];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                const uint32_t i = i0 + k;
                const uint32_t c = u4get(code_c, k);
                vtx[k] = c & kVMask;
                // SCC colouring: an assigned vertex holds INF (scc_init_kernel) and
                // breaks its paths -- the gathered master says so without a
                // second random load of its label
                live[k] = i >= wc.beg && i < wc.end && (MODE != 3 || a_c[k] != INF);
                hd[k] = !live[k] || (c & kHead);
                tl[k] = !live[k] || (c & kTail);
                wgt[k] = MODE == 0 ? (uint32_t)i4get(wv, k) : (MODE == 1 ? 1u : 0u);
                a[k] = live[k] ? a_c[k] : INF;
            }
            // lane aggregate of f_k(x) = hd ? a : min(a, x + w)
            bool H = false;
            uint32_t A = INF, W = 0;
#pragma unroll
            for (int k = 0; k < 4; k++) {
                if (hd[k]) { H = true; A = a[k]; W = 0; }
                else { A = min(a[k], sat_add(A, wgt[k])); W = sat_add(W, wgt[k]); }
            }
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {  // warp inclusive scan, prefix composed before self
                bool Hp = __shfl_up_sync(0xffffffffu, H, off);
                uint32_t Ap = __shfl_up_sync(0xffffffffu, A, off);
                uint32_t Wp = __shfl_up_sync(0xffffffffu, W, off);
                if (lane >= off && !H) { A = min(A, sat_add(Ap, W)); W = sat_add(Wp, W); H = Hp; }
            }
            bool He = __shfl_up_sync(0xffffffffu, H, 1);
            uint32_t Ae = __shfl_up_sync(0xffffffffu, A, 1);
            uint32_t We = __shfl_up_sync(0xffffffffu, W, 1);
            if (lane == 0) { He = false; Ae = INF; We = 0; }
            uint32_t cur = He ? Ae : min(Ae, sat_add(carry, We));
            uint32_t val[4];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                cur = hd[k] ? a[k] : min(a[k], sat_add(cur, wgt[k]));
                val[k] = cur;
            }
            if (MODE == 2) {
                // backward (suffix) min: x_i = min(a_i, x_(i+1)) until a tail
                bool T = false;
                uint32_t B = INF;
#pragma unroll
                for (int k = 3; k >= 0; k--) {
                    if (tl[k]) { T = true; B = a[k]; } else B = min(a[k], B);
                }
#pragma unroll
                for (int off = 1; off < 32; off <<= 1) {
                    bool Tn = __shfl_down_sync(0xffffffffu, T, off);
                    uint32_t Bn = __shfl_down_sync(0xffffffffu, B, off);
                    if (lane + off < 32 && !T) { B = min(B, Bn); T = Tn; }
                }
                uint32_t bc = __shfl_down_sync(0xffffffffu, B, 1);
                if (lane == 31) bc = nx_lab;
#pragma unroll
                for (int k = 3; k >= 0; k--) {
                    bc = tl[k] ? a[k] : min(a[k], bc);
                    val[k] = min(val[k], bc);
                }
            }
            bool changed3 = false;
            // path predecessor of entry 0 (previous lane's last entry, or the carry's vertex)
            uint32_t pred0 = __shfl_up_sync(0xffffffffu, vtx[3], 1);
            if (lane == 0) pred0 = carry_vtx;
            // the lane's (up to four) atomicMins are issued back to back and
            // are in flight together; their results are consumed afterwards
            uint32_t old[4];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                old[k] = 0u;
                if (live[k] && val[k] < a[k] && val[k] <= theta) old[k] = atomicMin(&P.vs_u[vtx[k]], val[k]);
            }
#pragma unroll
            for (int k = 0; k < 4; k++) {
                if (!live[k]) continue;
                acc.entries++;
                if (!(u4get(code_c, k) & kHead)) acc.edges++;
                if (val[k] < a[k]) {
                    if (val[k] > theta) {
                        // beyond this round's bucket: not committed; the path
                        // predecessor stays active so the edge is relaxed again
                        acc.sig += signal_vertex(bnxt, k ? vtx[k - 1] : pred0);
                        continue;
                    }
                    if (val[k] < old[k]) {
                        acc.upd++;
                        if (k == 3) changed3 = true;
                        // fire-and-forget signal (RED): the active counter may count a
                        // vertex lowered twice in one round twice -- an upper bound,
                        // which is all its uses need (non-zero test, sparse threshold)
                        atomicOr(&bnxt[vtx[k] >> 5], 1u << (vtx[k] & 31));
                        acc.sig++;
                        acc.vmin = min(acc.vmin, val[k]);
                    }
                }
            }
            // the carry into the next window is live if the path continues and its
            // last vertex changed now or was signalled (its out-edge must be relaxed)
            carry = __shfl_sync(0xffffffffu, cur, 31);
            carry_vtx = __shfl_sync(0xffffffffu, vtx[3], 31);
            carry_live = __shfl_sync(0xffffffffu, !tl[3] && (changed3 || act_c[3]), 31);
        } else {
            carry = INF;
            carry_live = false;
        }
        // rotate the pipeline
        wc = wn; wn = wn2; wn2 = wn3;
        code_c = code_n; code_n = code_n2; code_n2 = code_n3;
        words_n = words_n2;
        any_c = any_n;
#pragma unroll
        for (int k = 0; k < 4; k++) { act_c[k] = act_n[k]; a_c[k] = a_n[k]; }
    }
}

// Sparse min-plus rounds (SSSP/BFS, the forward half of WCC, SCC's forward
// colouring).  When few
// vertices are signalled, probing every window's signal bits costs more than
// the work: the round instead starts the path walks at the signalled vertices.
// Every out-edge of v lies on exactly one path, right after one of v's
// non-tail entries (the occurrence index), so walking forward from each
// occurrence relaxes exactly v's out-edges -- and, as in the dense walk, a
// vertex lowered on the way passes its new distance on along its path in the
// same round (the vertices of a path are handled in
// order and a new state is used immediately).  A walk stops at the path's
// tail, at a vertex it does not improve (that vertex's own distance was, or
// will be, propagated from its own signal), or at a relaxation beyond the
// round's bucket (reading R-DELTA: the predecessor stays signalled).
//
// Walks are capped at P.sparse_walk path edges: every vertex a walk lowers is
// signalled, so the walk's continuation is picked up in the next round; the
// cap bounds a round's latency (merged paths reach ~1000 edges).
//
// Frontier list: the round's signal bitmap compacted with warp-aggregated
// appends (one pass over n/32 words) into items (v, chunk) of at most
// kOccChunk occurrences, so a hub's out-edges spread over many warps.
constexpr uint32_t kOccChunk = 32;
// Pass 1 (count): out-edges and items of the signalled vertices.
__device__ void count_bits(const KParams& P, const uint32_t* off, const uint32_t* bcur, unsigned* qn, unsigned* osum) {
    const int64_t T = (int64_t)gridDim.x * blockDim.x;
    unsigned c = 0, o = 0;
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < P.nw; i += T) {
        for (uint32_t x = bcur[i]; x; x &= x - 1) {
            const uint32_t v = (uint32_t)(i * 32 + __ffs(x) - 1);
            const uint32_t d = off[v + 1] - off[v];
            c += (d + kOccChunk - 1) / kOccChunk;
            o += d;
        }
    }
    for (int sh = 16; sh; sh >>= 1) {
        c += __shfl_xor_sync(0xffffffffu, c, sh);
        o += __shfl_xor_sync(0xffffffffu, o, sh);
    }
    if ((threadIdx.x & 31) == 0 && o) {
        atomicAdd(qn, c);
        atomicAdd(osum, o);
    }
}
// Pass 2 (write): the items, appended warp by warp (order is irrelevant).
__device__ void compact_bits(const KParams& P, const uint32_t* off, const uint32_t* bcur, uint2* list, unsigned* cursor) {
    const int lane = threadIdx.x & 31;
    const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
    const int64_t gw = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
    for (int64_t b = gw * 32; b < P.nw; b += warps * 32) {
        const int64_t i = b + lane;
        uint32_t w = i < P.nw ? bcur[i] : 0u;
        unsigned c = 0;
        for (uint32_t x = w; x; x &= x - 1) {
            const uint32_t v = (uint32_t)(i * 32 + __ffs(x) - 1);
            c += (off[v + 1] - off[v] + kOccChunk - 1) / kOccChunk;
        }
        unsigned inc = c;
#pragma unroll
        for (int sh = 1; sh < 32; sh <<= 1) {
            const unsigned y = __shfl_up_sync(0xffffffffu, inc, sh);
            if (lane >= sh) inc += y;
        }
        const unsigned tot = __shfl_sync(0xffffffffu, inc, 31);
        if (tot == 0) continue;
        unsigned base = 0;
        if (lane == 31) base = atomicAdd(cursor, tot);
        base = __shfl_sync(0xffffffffu, base, 31) + inc - c;
        while (w) {
            const uint32_t v = (uint32_t)(i * 32 + __ffs(w) - 1);
            w &= w - 1;
            const uint32_t nch = (off[v + 1] - off[v] + kOccChunk - 1) / kOccChunk;
            for (uint32_t k = 0; k < nch; k++) list[base++] = make_uint2(v, k);
        }
    }
}
// A round's sparse decision: few signalled vertices whose out-edges are at
// most M / sparse_div; a sparse round compacts the frontier into P.occ_items.
// (Counting at the end of the previous round, folded into its last barrier,
// and compacting there were both measured: no gain / slower.)
__device__ bool sparse_round(const KParams& P, cg::grid_group& grid, int cur, const uint32_t* bcur) {
    if (!P.occ_off || *((volatile unsigned*)&P.ctr->active[cur]) > P.sparse_max) return false;
    count_bits(P, P.occ_off, bcur, &P.ctr->qn[cur], &P.ctr->osum[cur]);
    grid.sync();
    if (*((volatile unsigned*)&P.ctr->osum[cur]) > P.sparse_occ) return false;
    compact_bits(P, P.occ_off, bcur, P.occ_items, &P.ctr->qcur[cur]);
    grid.sync();
    return true;
}

template <int MODE>
__device__ void walk_sparse(const KParams& P, const uint32_t* off, const uint32_t* occ, const uint2* list, unsigned qn,
                            unsigned* ticket, uint32_t* bnxt,
                            uint32_t theta, Acc& acc) {
    __shared__ uint32_t s_off[kWarps][33];
    __shared__ uint32_t s_beg[kWarps][32], s_x[kWarps][32], s_v[kWarps][32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    while (true) {
        unsigned t = 0;
        if (lane == 0) t = atomicAdd(ticket, 32u);
        t = __shfl_sync(0xffffffffu, t, 0);
        if (t >= qn) break;
        uint32_t cnt = 0, beg = 0, x = INF, v = 0;
        if (t + lane < qn) {
            const uint2 it = list[t + lane];
            v = it.x;
            beg = off[v] + it.y * kOccChunk;
            cnt = min(off[v + 1] - beg, kOccChunk);
            x = P.vs_u[v];
            acc.units++;
        }
        uint32_t inc = cnt;
#pragma unroll
        for (int sh = 1; sh < 32; sh <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, sh);
            if (lane >= sh) inc += y;
        }
        s_off[wid][lane + 1] = inc;
        if (lane == 0) s_off[wid][0] = 0;
        s_beg[wid][lane] = beg;
        s_x[wid][lane] = x;
        s_v[wid][lane] = v;
        __syncwarp();
        const uint32_t total = s_off[wid][32];
        for (uint32_t j = lane; j < total; j += 32) {
            int lo = 0, hi = 31;  // owner: largest o with s_off[o] <= j
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (s_off[wid][mid] <= j) lo = mid; else hi = mid - 1;
            }
            uint32_t cur = s_x[wid][lo], pred = s_v[wid][lo];
            uint32_t e = occ[s_beg[wid][lo] + (j - s_off[wid][lo])] + 1;  // the path edge out of the occurrence
            // the next entry of the path is loaded one step ahead
            uint32_t code, w;
            if (MODE == 0 && P.e_cw) {  // one random 8-byte load per step instead of two 4-byte ones
                const uint2 cw = __ldg(P.e_cw + e);
                code = cw.x;
                w = cw.y;
            } else {
                code = __ldg(P.e_idx + e);
                w = MODE == 0 ? (uint32_t)__ldg(P.e_w + e) : (MODE == 1 ? 1u : 0u);
            }
            for (int step = 0; step < P.sparse_walk; step++) {
                const uint32_t u = code & kVMask;
                // the head's state, read once (before the atomic: in-edges of hubs
                // would otherwise serialise on one address); SCC colouring: an
                // assigned vertex holds INF and breaks its paths
                const uint32_t cu = __ldcg(&P.vs_u[u]);
                if (MODE == 3 && cu == INF) break;
                const uint32_t cand = MODE == 3 ? cur : sat_add(cur, w);
                const bool last = code & kTail;
                acc.entries++;
                acc.edges++;
                if (cand > theta) {  // beyond the bucket: not committed, the predecessor stays signalled
                    acc.sig += signal_vertex(bnxt, pred);
                    break;
                }
                // when even a weight-1 relaxation after this entry would lie
                // beyond the bucket, the walk ends here -- the vertex it lowers
                // is signalled and relaxes its edges in a later round (no wasted
                // load of the next entry, no redundant re-signal; a 0-weight
                // continuation is merely deferred, which label correction allows)
                const bool stop_next = (MODE == 0 || MODE == 1) && sat_add(cand, 1u) > theta;
                if (!last && !stop_next) {  // prefetch the path's next entry
                    if (MODE == 0 && P.e_cw) {
                        const uint2 cw = __ldg(P.e_cw + e + 1);
                        code = cw.x;
                        w = cw.y;
                    } else {
                        code = __ldg(P.e_idx + e + 1);
                        if (MODE == 0) w = (uint32_t)__ldg(P.e_w + e + 1);
                    }
                }
                if (cand >= cu) break;
                const uint32_t old = atomicMin(&P.vs_u[u], cand);
                if (cand >= old) break;
                acc.upd++;
                acc.sig += signal_vertex(bnxt, u);
                acc.vmin = min(acc.vmin, cand);
                if (last || stop_next) break;
                cur = cand;
                pred = u;
                e++;
            }
        }
        __syncwarp();
    }
}

// Sparse backward rounds of the SCC reachability phase: from each marked
// vertex v, walk its in-edges backwards (P.occ_off/P.occ hold the non-head
// entries here: the path edge INTO entry i comes from entry i-1) and mark
// unassigned predecessors of v's colour, passing the mark on along the path.
// WCC: the same backward walk carries the smallest label (atomicMin) instead.
template <bool WCC>
__device__ void walk_sparse_bwd(const KParams& P, const uint32_t* off, const uint32_t* occ, const uint2* list,
                                unsigned qn, unsigned* ticket, uint32_t* bnxt, Acc& acc) {
    __shared__ uint32_t s_off[kWarps][33];
    __shared__ uint32_t s_beg[kWarps][32], s_x[kWarps][32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    while (true) {
        unsigned t = 0;
        if (lane == 0) t = atomicAdd(ticket, 32u);
        t = __shfl_sync(0xffffffffu, t, 0);
        if (t >= qn) break;
        uint32_t cnt = 0, beg = 0, col = INF;
        if (t + lane < qn) {
            const uint2 it = list[t + lane];
            beg = off[it.x] + it.y * kOccChunk;
            cnt = min(off[it.x + 1] - beg, kOccChunk);
            col = P.vs_u[it.x];
            acc.units++;
        }
        uint32_t inc = cnt;
#pragma unroll
        for (int sh = 1; sh < 32; sh <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, sh);
            if (lane >= sh) inc += y;
        }
        s_off[wid][lane + 1] = inc;
        if (lane == 0) s_off[wid][0] = 0;
        s_beg[wid][lane] = beg;
        s_x[wid][lane] = col;
        __syncwarp();
        const uint32_t total = s_off[wid][32];
        for (uint32_t j = lane; j < total; j += 32) {
            int lo = 0, hi = 31;
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (s_off[wid][mid] <= j) lo = mid; else hi = mid - 1;
            }
            const uint32_t c = s_x[wid][lo];
            uint32_t e = occ[s_beg[wid][lo] + (j - s_off[wid][lo])] - 1;  // the path predecessor
            for (int step = 0; step < P.sparse_walk; step++) {
                const uint32_t code = __ldg(P.e_idx + e);
                const uint32_t u = code & kVMask;
                acc.entries++;
                acc.edges++;
                if (WCC) {
                    if (c >= __ldcg(&P.vs_u[u]) || c >= atomicMin(&P.vs_u[u], c)) break;
                    acc.upd++;
                    acc.sig += signal_vertex(bnxt, u);
                } else {
                    if (P.vs_u[u] != c || P.mark[u]) break;  // assigned vertices hold INF != c
                    P.mark[u] = 1;  // idempotent byte store; the signal bit counts it once
                    if (signal_vertex(bnxt, u)) {
                        acc.upd++;
                        acc.sig++;
                    }
                }
                if (code & kHead) break;
                e--;
            }
        }
        __syncwarp();
    }
}

// Accumulative walk (PageRank / Adsorption; DESIGN.md "Accumulative
// propagation").  Every vertex keeps its accumulated total T (the master,
// V_val of PAPER.md Fig. 4) and every non-tail entry i keeps the mirror
// S_val[i] = the part of T(v_i) already pushed along the path edge out of i.
// Walking a path in order, entry i pushes
//     a_i = c_i * (pend_i + p_i),   pend_i = T_i - S_val[i] if >= eps else 0,
// where p_i = a_(i-1) is what its path predecessor pushed in this same walk
// (used immediately, Observation 1) and c_i the path edge's coefficient
// (d/outdeg for PageRank, streamed per entry).  p_i is added to T(v_i) and
// S_val[i] += pend_i + p_i.  T and S_val are exact 64-bit fixed point (2^-32
// units; reading R-FX): pend is an exact difference and conversions
// truncate, so no push is inflated by rounding and every cycle contracts --
// fp32 totals livelock once eps is ~1 ulp of T.  A window is walked when one
// of its entries has pend >= eps or a path carries a push into it.
constexpr float kFxScale = 4294967296.0f;          // 2^32
constexpr float kFxInv = 2.3283064365386963e-10f;  // 2^-32
__device__ __forceinline__ unsigned long long fx_from(float x) { return x > 0.f ? __float2ull_rz(x * kFxScale) : 0ull; }
__device__ __forceinline__ float fx_to(unsigned long long v) { return __ull2float_rn(v) * kFxInv; }

// Shared-memory proxies of the n_proxy highest-degree vertices (internal ids
// [0, H)): "creates a proxy vertex in the shared memory of
// each related SMX for each vertex with high in-degree, to accumulate the
// pushed new states of its local mirrors ... sent to the master when the
// partition assigned to this SMX has been handled".  Per CTA: the round-start
// totals and the CTA's unflushed pushes.
// The pushes accumulate in two 32-bit words per hub (lo, hi) because shared
// memory has native 32-bit atomic adds only (a 64-bit add is a CAS loop): lo
// takes the push, its carry goes to hi.  A concurrent reader can see a carry
// not yet applied (an under-estimate: pend only shrinks, safe) and a flush can
// leave a pending carry for the next flush (the total is conserved).
// (Measured against write-only proxies with three 16-bit limbs and fire-and-
// forget shared REDs: no faster.)
struct Proxies {
    unsigned long long* T;  // snapshot of the hub totals
    unsigned* acc;          // 2 words per hub
    int64_t H;
};
__device__ __forceinline__ void px_add(unsigned* a, unsigned long long p) {
    const unsigned lo = (unsigned)p, hi = (unsigned)(p >> 32);
    const unsigned old = atomicAdd(&a[0], lo);
    const unsigned c = hi + (old + lo < old ? 1u : 0u);
    if (c) atomicAdd(&a[1], c);
}
__device__ __forceinline__ unsigned long long px_read(const unsigned* a) {
    const unsigned lo = *(const volatile unsigned*)&a[0], hi = *(const volatile unsigned*)&a[1];
    return ((unsigned long long)hi << 32) + lo;
}
__device__ __forceinline__ unsigned long long px_take(unsigned* a) {
    const unsigned lo = atomicExch(&a[0], 0u), hi = atomicExch(&a[1], 0u);
    return ((unsigned long long)hi << 32) + lo;
}
constexpr int kPxBytes = 16;  // shared memory per proxied hub

// Mid-round proxy flush (every px_refresh partitions a CTA starts): one warp
// sends the proxies' accumulated pushes to the masters and reloads the
// snapshot, so hub totals propagate between CTAs within the round.  The
// reloads are batched (16 L2 loads in flight per lane).
__device__ __forceinline__ void px_refresh(const KParams& P, const Proxies& px) {
    const int lane = threadIdx.x & 31;
    for (int64_t i = lane; i < px.H; i += 32) {
        const unsigned long long a = px_take(&px.acc[2 * i]);
        if (a) atomicAdd(&P.vs_t[i], a);
    }
    __syncwarp();
    for (int64_t i0 = lane; i0 < px.H; i0 += 32 * 16) {
        unsigned long long t16[16];
#pragma unroll
        for (int u = 0; u < 16; u++) t16[u] = i0 + 32 * u < px.H ? __ldcg(&P.vs_t[i0 + 32 * u]) : 0ull;
#pragma unroll
        for (int u = 0; u < 16; u++)
            if (i0 + 32 * u < px.H) px.T[i0 + 32 * u] = t16[u];
    }
}

// Walk all windows the warp obtains in this round.  Software pipeline over the
// window stream (kRing-slot shared ring per warp): while window w is walked,
// the master totals of windows w+1 and w+2 are in flight into shared memory
// (cp.async: no registers held), the mirrors and coefficients of window w+1
// into registers, and the indices of window w+3.  Reading a master two
// windows early is a read slightly before the walk reaches it -- the same
// asynchronous semantics as any concurrent push.
constexpr int kRing = 3;
template <int NW>
__host__ __device__ constexpr size_t gbuf_bytes() { return (size_t)NW * kRing * 128 * sizeof(uint4); }
template <bool ADS>
__device__ void walk_accum(const KParams& P, const Queue& q, Acc& acc, unsigned long long pol_stream,
                           unsigned long long pol_keep, const Proxies& px, uint4* gbuf, int* s_done) {
    const int lane = threadIdx.x & 31;
    const unsigned long long eps = P.eps_fx;
    const uint4 kFill = make_uint4(kHead | kTail, kHead | kTail, kHead | kTail, kHead | kTail);
    auto load_code = [&](const Win& w) {
        uint4 c = kFill;
        if (w.base != kNoWin && w.base + 4 * lane < w.end) c = ld_stream_u4_h(P.e_idx + w.base + 4 * lane, pol_stream);
        return c;
    };
    auto load_sv = [&](const Win& w, unsigned long long (&sv)[4], float4& cf) {
        if (w.base != kNoWin && w.base + 4 * lane < w.end && !EXP_ON(P, 16)) {
            ld_stream_u64x4_h(P.s_val + w.base + 4 * lane, sv, pol_stream);
            cf = ld_stream_f4_h(P.e_coef + w.base + 4 * lane, pol_stream);
        } else {
            sv[0] = sv[1] = sv[2] = sv[3] = 0ull;
            cf = make_float4(0.f, 0.f, 0.f, 0.f);
        }
    };
    // masters of a window into ring slot s: entry 4*lane+k -> gbuf[s*128 + k*32 + lane]
    // (16-byte aligned pair {T[v & ~1], T[v | 1]}); proxies, tails (no out-edge:
    // nothing pending to forward) and invalid entries skip
    auto gather = [&](const Win& w, const uint4& code, int s) {
        if (w.base != kNoWin) {
#pragma unroll
            for (int k = 0; k < 4; k++) {
                const uint32_t i = w.base + 4 * lane + k;
                const uint32_t c = u4get(code, k);
                const uint32_t v = c & kVMask;
                if (i >= w.beg && i < w.end && v >= px.H && !(c & kTail) && !EXP_ON(P, 2))
                    cp_async16(&gbuf[s * 128 + k * 32 + lane],
                               (EXP_ON(P, 96) ? P.snap + (size_t)((P.n + 3) & ~1ll) * *(volatile int*)&g_exp_par : P.vs_t) + (v & ~1u),
                               pol_keep);
            }
        }
        cp_async_commit();
    };

    Feed f{0u, kNoWin, 0u};
    Win w0 = feed_start(P, q, f);
    if (w0.base == kNoWin) return;
    Win w1 = feed_next(P, q, w0, f);
    Win w2 = feed_next(P, q, w1, f);
    uint4 c0 = load_code(w0), c1 = load_code(w1), c2 = load_code(w2);
    unsigned long long sv_c[4], sv_n[4];
    float4 cf_c, cf_n;
    load_sv(w0, sv_c, cf_c);
    gather(w0, c0, 0);
    gather(w1, c1, 1);
    int slot = 0;
    float carry = 0.f;
    while (w0.base != kNoWin) {
        const Win w3 = feed_next(P, q, w2, f);
        const uint4 c3 = load_code(w3);
        gather(w2, c2, slot == 0 ? 2 : slot - 1);  // slot (w+2) % kRing
        load_sv(w1, sv_n, cf_n);
        const bool part_start = w0.base == (w0.beg & ~3u);
        if (part_start) {
            carry = 0.f;
            if (px.H && P.px_refresh > 0) {
                int c = 0;
                if (lane == 0) c = atomicAdd(s_done, 1) + 1;
                c = __shfl_sync(0xffffffffu, c, 0);
                if (c % P.px_refresh == 0) px_refresh(P, px);
            }
        }
        asm volatile("cp.async.wait_group 2;" ::: "memory");  // window w's masters (its own lane's copies)
        const uint32_t i0 = w0.base + 4 * lane;
        uint32_t vtx[4];
        unsigned long long T[4], pend[4];
        bool valid[4], hd[4], tl[4], any_act = false;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t i = i0 + k;
            const uint32_t c = u4get(c0, k);
            valid[k] = i >= w0.beg && i < w0.end;
            vtx[k] = c & kVMask;
            hd[k] = !valid[k] || (c & kHead);
            tl[k] = !valid[k] || (c & kTail);
            T[k] = 0ull;
            if (valid[k]) {
                if (vtx[k] < px.H) {
                    T[k] = px.T[vtx[k]] + px_read(&px.acc[2 * vtx[k]]);
                } else {
                    const uint4 g = gbuf[slot * 128 + k * 32 + lane];
                    T[k] = (vtx[k] & 1u) ? ((unsigned long long)g.w << 32 | g.z) : ((unsigned long long)g.y << 32 | g.x);
                }
            }
            const unsigned long long pd = T[k] > sv_c[k] ? T[k] - sv_c[k] : 0ull;
            pend[k] = (!tl[k] && pd >= eps) ? pd : 0ull;
            any_act |= pend[k] != 0ull;
        }
        if (__any_sync(0xffffffffu, any_act) || carry != 0.f) {
            acc.units++;
            float al[4], be[4];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                const float coef = f4get(cf_c, k);
                al[k] = tl[k] ? 0.f : coef * fx_to(pend[k]);
                be[k] = (tl[k] || hd[k]) ? 0.f : coef;
            }
            // in-order walk = inclusive warp scan of the entries' affine maps
            // p_(i+1) = al_i + be_i * p_i (heads reset, tails push nothing)
            float Al = 0.f, Be = 1.f;
#pragma unroll
            for (int k = 0; k < 4; k++) { Al = al[k] + be[k] * Al; Be = be[k] * Be; }
#pragma unroll
            for (int off = 1; off < 32; off <<= 1) {
                const float Ap = __shfl_up_sync(0xffffffffu, Al, off);
                const float Bp = __shfl_up_sync(0xffffffffu, Be, off);
                if (lane >= off) { Al = Al + Be * Ap; Be = Be * Bp; }
            }
            float Ae = __shfl_up_sync(0xffffffffu, Al, 1);
            float Bx = __shfl_up_sync(0xffffffffu, Be, 1);
            if (lane == 0) { Ae = 0.f; Bx = 1.f; }
            float prev = Ae + Bx * carry;
            float pin[4];
#pragma unroll
            for (int k = 0; k < 4; k++) {
                pin[k] = hd[k] ? 0.f : prev;
                prev = al[k] + be[k] * prev;
            }
            carry = __shfl_sync(0xffffffffu, prev, 31);
            bool dirty = false;
            unsigned n_valid = 0, n_edges = 0, n_upd = 0;
#pragma unroll
            for (int k = 0; k < 4; k++) {
                if (!valid[k]) continue;
                n_valid++;
                n_edges += !hd[k];
                const unsigned long long p = fx_from(pin[k]);
                if (p) {
                    if (vtx[k] < px.H) px_add(&px.acc[2 * vtx[k]], p);  // proxy: shared-memory atomics
                    else if (!EXP_ON(P, 1)) red_add_u64_h(&P.vs_t[vtx[k]], p, pol_keep);  // master: REDG (no return)
                    n_upd++;
                }
                if (!tl[k] && (pend[k] | p)) { sv_c[k] += pend[k] + p; dirty = true; }
            }
            acc.entries += n_valid;
            acc.edges += n_edges;
            acc.upd += n_upd;
            // lanes whose four entries all lie in this partition write one 256-bit
            // store; lanes at the partition's ends write only their own entries
            // (the neighbouring partition's mirrors belong to another warp)
            if (dirty && !EXP_ON(P, 4)) {
                if (i0 >= w0.beg && i0 + 3 < w0.end) {
                    st_stream_u64x4_h(P.s_val + i0, sv_c, pol_stream);
                } else {
#pragma unroll
                    for (int k = 0; k < 4; k++)
                        if (valid[k]) st_stream_u64_h(P.s_val + i0 + k, sv_c[k], pol_stream);
                }
            }
        } else {
            carry = 0.f;
        }
        // rotate the pipeline
        w0 = w1; w1 = w2; w2 = w3;
        c0 = c1; c1 = c2; c2 = c3;
#pragma unroll
        for (int k = 0; k < 4; k++) sv_c[k] = sv_n[k];
        cf_c = cf_n;
        slot = slot == kRing - 1 ? 0 : slot + 1;
    }
    cp_async_wait0();
    // an unused prefetched ticket is simply dropped (the round's ticket only
    // needs to exceed n_part, which it then does)
}

// End-of-round vertex sweep of the accumulative algorithms: a vertex whose
// total grew by >= eps since its last signal counts as signalled for the next
// round (the per-vertex stop rule at delta < eps; the device active counter).
// The signalled vertices also form the next round's bitmap (whole words: a
// warp sweeps 32 consecutive vertices), read by sparse rounds.
__device__ void accum_sweep(const KParams& P, uint32_t* bnxt, unsigned& cnt) {
    const int64_t stride = (int64_t)gridDim.x * blockDim.x;
    for (int64_t v0 = blockIdx.x * (int64_t)blockDim.x; v0 < P.n; v0 += stride) {
        const int64_t v = v0 + threadIdx.x;
        bool sig = false;
        if (v < P.n) {
            const unsigned long long T = __ldcg(&P.vs_t[v]);
            if (T - P.sigma[v] >= P.eps_fx) {
                P.sigma[v] = T;
                cnt++;
                sig = true;
            }
        }
        const unsigned word = __ballot_sync(0xffffffffu, sig);
        if ((threadIdx.x & 31) == 0 && v < P.n + 31) bnxt[v >> 5] = word;
    }
}

// Sparse accumulative rounds (PageRank / Adsorption; DESIGN.md "Sparse
// rounds").  From every non-tail entry i of a signalled vertex the walk
// forwards pend_i (if >= eps) along the path edge out of i exactly as the
// dense walk does, and passes the push on along the path: at entry e of
// vertex x with incoming push p it reads T(x), adds p to T(x) (RED), forwards
// c_e * (pend_e + p) and sets S_val[e] += pend_e + p.  Each entry has a single
// owner in a round (as in the dense walk, where a warp owns a window): the
// starter at a signalled vertex's entry, or the walk arriving from the path
// predecessor when the entry's vertex is not signalled.  A walk arriving at a
// signalled vertex's entry (that entry has its own starter), at a tail, or at
// the length cap only adds its push to the master; the push stays pending in
// T(x) - S_val[e], like any push from another path.
template <int NW>
__device__ void walk_sparse_acc(const KParams& P, const uint2* list, unsigned qn, unsigned* ticket,
                                const uint32_t* bcur, Acc& acc) {
    __shared__ uint32_t s_off[NW][33];
    __shared__ uint32_t s_beg[NW][32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const unsigned long long eps = P.eps_fx;
    while (true) {
        unsigned t = 0;
        if (lane == 0) t = atomicAdd(ticket, 32u);
        t = __shfl_sync(0xffffffffu, t, 0);
        if (t >= qn) break;
        uint32_t cnt = 0, beg = 0;
        if (t + lane < qn) {
            const uint2 it = list[t + lane];
            beg = P.occ_off[it.x] + it.y * kOccChunk;
            cnt = min(P.occ_off[it.x + 1] - beg, kOccChunk);
            acc.units++;
        }
        uint32_t inc = cnt;
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, off);
            if (lane >= off) inc += y;
        }
        s_off[wid][lane + 1] = inc;
        if (lane == 0) s_off[wid][0] = 0;
        s_beg[wid][lane] = beg;
        __syncwarp();
        const uint32_t total = s_off[wid][32];
        for (uint32_t j = lane; j < total; j += 32) {
            int lo = 0, hi = 31;
            while (lo < hi) {
                const int mid = (lo + hi + 1) >> 1;
                if (s_off[wid][mid] <= j) lo = mid; else hi = mid - 1;
            }
            uint32_t e = P.occ[s_beg[wid][lo] + (j - s_off[wid][lo])];
            uint32_t x = __ldg(P.e_idx + e) & kVMask;
            unsigned long long p = 0ull;  // push arriving at entry e
            for (int step = 0; step <= P.sparse_walk; step++) {
                const uint32_t code = step ? __ldg(P.e_idx + e) : 0u;
                const unsigned long long T = __ldcg(&P.vs_t[x]);
                if (p) {
                    atomicAdd(&P.vs_t[x], p);
                    acc.upd++;
                }
                acc.entries++;
                if (step) acc.edges++;
                // stop: tail, the entry has its own starter, or the cap (the push stays pending)
                if (step && ((code & kTail) || test_bit(bcur, x) || step == P.sparse_walk)) break;
                const unsigned long long sv = P.s_val[e];
                const unsigned long long pd = T > sv ? T - sv : 0ull;
                const unsigned long long amt = (pd >= eps ? pd : 0ull) + p;
                if (!amt) break;
                P.s_val[e] = sv + amt;
                p = fx_from(__ldg(P.e_coef + e) * fx_to(amt));
                if (!p) break;
                e++;
                x = __ldg(P.e_idx + e) & kVMask;
            }
        }
        __syncwarp();
    }
}

// SCC backward reachability inside a colour: walking every
// path backwards, mark_i |= mark_(i+1) when both are unassigned and share the
// colour.  Windows are walked from the partition's end to its start so the
// suffix carry crosses windows.
__device__ void walk_scc_bwd(const KParams& P, int64_t beg, int64_t end, const uint32_t* bcur, uint32_t* bnxt,
                             Acc& acc) {
    const int lane = threadIdx.x & 31;
    bool carry = false, carry_live = false;  // mark of the entry after the window
    uint32_t carry_col = INF;                // its colour (INF: none / tail boundary)
    const int64_t first = beg & ~(int64_t)3;
    const int64_t nwin = (end - first + 127) / 128;
    for (int64_t wi = nwin - 1; wi >= 0; wi--) {
        const int64_t base = first + wi * 128;
        const int64_t i0 = base + 4 * lane;
        uint4 code = make_uint4(kHead | kTail, kHead | kTail, kHead | kTail, kHead | kTail);
        if (i0 < end) code = ld_stream_u4(P.e_idx + i0);
        uint32_t vtx[4];
        bool valid[4], act[4], any_act = false;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const int64_t i = i0 + k;
            valid[k] = i >= beg && i < end;
            vtx[k] = u4get(code, k) & kVMask;
            act[k] = valid[k] && test_bit(bcur, vtx[k]);
            any_act |= act[k];
        }
        if (!__any_sync(0xffffffffu, any_act) && !carry_live) {
            // this window's first entry is the next window's successor: not marked newly
            carry = false; carry_col = INF; carry_live = false;
            continue;
        }
        acc.units++;
        uint32_t col[4];
        bool tl[4], live[4], mk[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t c = u4get(code, k);
            // an assigned vertex holds INF (scc_init_kernel): its colour says
            // it breaks the path, without a load of its label
            const uint32_t cv = valid[k] ? P.vs_u[vtx[k]] : INF;
            live[k] = cv != INF;
            tl[k] = !live[k] || (c & kTail);
            col[k] = cv;
            mk[k] = live[k] && P.mark[vtx[k]];
        }
        // element k on the successor's mark x:  m_k = mk_k | (x & eq_k),
        // eq_k = !tl_k && col_k == col_(k+1).  Represented as f(x) = O | (Q & x).
        uint32_t col_next_lane = __shfl_down_sync(0xffffffffu, col[0], 1);
        if (lane == 31) col_next_lane = carry_col;
        bool O[4], Q[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const uint32_t cn = k < 3 ? col[k + 1] : col_next_lane;
            Q[k] = !tl[k] && col[k] == cn && cn != INF;
            O[k] = mk[k];
        }
        bool AO = false, AQ = true;
#pragma unroll
        for (int k = 3; k >= 0; k--) { AO = O[k] | (Q[k] & AO); AQ = Q[k] & AQ; }
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {  // warp suffix scan
            bool On = __shfl_down_sync(0xffffffffu, AO, off);
            bool Qn = __shfl_down_sync(0xffffffffu, AQ, off);
            if (lane + off < 32) { AO = AO | (AQ & On); AQ = AQ & Qn; }
        }
        bool Oe = __shfl_down_sync(0xffffffffu, AO, 1);
        bool Qe = __shfl_down_sync(0xffffffffu, AQ, 1);
        if (lane == 31) { Oe = false; Qe = true; }
        bool x = Oe | (Qe & carry);
        bool newm[4];
#pragma unroll
        for (int k = 3; k >= 0; k--) {
            x = O[k] | (Q[k] & x);
            newm[k] = x;
        }
        bool changed0 = false;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            if (!live[k]) continue;
            acc.entries++;
            if (!tl[k]) acc.edges++;
            if (newm[k] && !mk[k]) {
                P.mark[vtx[k]] = 1;  // idempotent byte store
                acc.upd++;
                acc.sig += signal_vertex(bnxt, vtx[k]);
                if (k == 0) changed0 = true;
            }
        }
        carry = __shfl_sync(0xffffffffu, newm[0], 0);
        carry_col = __shfl_sync(0xffffffffu, col[0], 0);
        carry_live = __shfl_sync(0xffffffffu, newm[0] && (changed0 || act[0]), 0);
    }
}

// ------------------------------------------------------------------ persistent round driver
// Dynamic shared memory of the accumulative kernels: the per-warp kRing x
// 128-entry master rings (kAccWarps x 6 KB), then the CTA's proxies (16 B per
// hub).  The accumulative kernels run ONE CTA of kAccWarps warps per SM, so
// the SM's shared memory holds one proxy table (not one per CTA).
constexpr int kAccWarps = 16;

// ---- fused multi-rank exchange (P.mr.world > 1; DESIGN.md "Peer-memory
// exchange"): the same protocol as dg_boundary_exchange, run by the
// persistent kernel between rounds, plus the global termination test.
// Exchange e: every thread packs boundary values into this rank's slot e&1
// and counts the ones that differ from the last exchange's result; warp 0 of
// block 0 publishes (activity = signalled vertices + changed boundary values)
// and epoch e to every peer, waits for every peer's epoch e and sums their
// activities; every thread then reduces all ranks' slot e&1 into its masters
// (signalling changed vertices into bitmap ncur).  Activity 0 on every rank
// means no rank has work and no boundary value changed since the last
// exchange -- the reduction cannot change anything: the run is converged.
__device__ __forceinline__ bool mr_exchange(const KParams& P, cg::grid_group& grid, int ncur, unsigned long long e) {
    const MultiRank& M = P.mr;
    const int lane = threadIdx.x & 31;
    const int64_t T = (int64_t)gridDim.x * blockDim.x, t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const size_t off = kP2PHeader + (size_t)(e & 1) * M.slot_bytes;
    unsigned long long* mine = (unsigned long long*)((unsigned char*)M.own + off);
    unsigned dirty = 0;
    // only the ranks holding a boundary vertex take part in its reduction: a
    // rank packs and reduces the vertices its paths hold, reading the slots of
    // their other holders only (DESIGN.md sec. 4 "Peer-memory exchange")
    for (int64_t k = t0; k < M.nb; k += T) {
        if (!((M.hold[k] >> M.rank) & 1ull)) continue;
        const int v = M.bnd[k];
        if (M.sum) {
            const unsigned long long g = P.vs_t[v] - M.base[k];
            mine[k] = g;
            dirty += g != 0;
        } else {
            const uint32_t x = M.mark ? (P.mark[v] ? 0u : 1u) : P.vs_u[v];
            mine[k] = x;
            dirty += x != M.last[k];
        }
    }
    for (int sh = 16; sh; sh >>= 1) dirty += __shfl_xor_sync(0xffffffffu, dirty, sh);
    if (lane == 0 && dirty) atomicAdd(&P.ctr->mr_dirty, (unsigned long long)dirty);
    grid.sync();
    if (blockIdx.x == 0 && threadIdx.x < 32) {
        const int q = lane;
        if (q == 0) {
            const unsigned long long act = *((volatile unsigned*)&P.ctr->active[ncur]) +
                                           *((volatile unsigned long long*)&P.ctr->mr_dirty);
            *((volatile unsigned long long*)&M.own[kP2PCount + (e & 1)]) = act;
            P.ctr->mr_dirty = 0;
            __threadfence_system();
        }
        __syncwarp();
        if (q < M.world && q != M.rank) {
            __threadfence_system();
            unsigned long long* f = (unsigned long long*)M.region[q] + M.rank;
            asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(e) : "memory");
        }
        bool late = false;
        unsigned long long c = 0;
        if (q < M.world && q != M.rank) {
            unsigned long long ts, t, v;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(ts));
            while (true) {
                asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(M.own + q) : "memory");
                if (v >= e) break;
                asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
                if (t - ts > M.timeout_ns) { late = true; break; }
                __nanosleep(256);
            }
            const unsigned long long* pc = (const unsigned long long*)M.region[q] + kP2PCount + (e & 1);
            asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(c) : "l"(pc) : "memory");
        } else if (q == M.rank) {
            c = *((volatile unsigned long long*)&M.own[kP2PCount + (e & 1)]);
        }
        for (int sh = 16; sh; sh >>= 1) c += __shfl_xor_sync(0xffffffffu, c, sh);
        const bool any_late = __any_sync(0xffffffffu, late);
        if (q == 0) {
            P.ctr->mr_total = any_late ? 0ull : c;
            if (any_late) P.ctr->mr_err = 1;
        }
    }
    grid.sync();
    if (*((volatile unsigned long long*)&P.ctr->mr_err)) return true;
    uint32_t* b = P.bits + (int64_t)ncur * P.nw;
    unsigned cnt = 0;
    for (int64_t k = t0; k < M.nb; k += T) {
        const unsigned long long hm = M.hold[k];
        if (!((hm >> M.rank) & 1ull)) continue;
        const int v = M.bnd[k];
        if (M.sum) {
            unsigned long long g = 0;
            for (unsigned long long q = hm; q; q &= q - 1)
                g += __ldcv((const unsigned long long*)(M.region[__ffsll((long long)q) - 1] + off) + k);
            const unsigned long long t = M.base[k] + g;
            M.base[k] = t;
            P.vs_t[v] = t;
            if (t - P.sigma[v] >= M.eps_fx) {
                P.sigma[v] = t;
                cnt += signal_vertex(b, (uint32_t)v);
            }
        } else {
            unsigned long long m = ~0ull;
            for (unsigned long long q = hm; q; q &= q - 1)
                m = min(m, __ldcv((const unsigned long long*)(M.region[__ffsll((long long)q) - 1] + off) + k));
            M.last[k] = (uint32_t)m;
            if (M.mark) {  // marked on some rank: reachable backward from its colour's root
                if (m == 0 && !P.mark[v] && P.scc_label[v] < 0) {
                    P.mark[v] = 1;
                    cnt += signal_vertex(b, (uint32_t)v);
                }
            } else if ((uint32_t)m < P.vs_u[v]) {
                P.vs_u[v] = (uint32_t)m;
                cnt += signal_vertex(b, (uint32_t)v);
            }
        }
    }
    for (int sh = 16; sh; sh >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, sh);
    if (lane == 0 && cnt) atomicAdd(&P.ctr->active[ncur], cnt);
    grid.sync();
    return *((volatile unsigned long long*)&P.ctr->mr_total) == 0;
}

// MR: fused multi-rank run (P.mr.world > 1) -- a separate instantiation, so a
// single-rank run carries none of its code or registers
template <int ALGO, int MINB = DG_PATH_MINB, bool MR = false,
          int NW = (ALGO == DG_PAGERANK || ALGO == DG_ADSORPTION) ? kAccWarps : kWarps>
__global__ void __launch_bounds__(NW * 32, MINB) path_kernel(KParams P) {
    cg::grid_group grid = cg::this_grid();
    const int lane = threadIdx.x & 31;
    constexpr bool kAccum = ALGO == DG_PAGERANK || ALGO == DG_ADSORPTION;
    const unsigned long long pol_stream = policy_evict_first();
    unsigned long long pol_keep = policy_evict_last();
    if (kAccum) {  // masters: hot prefix evict-last (at most kHotMasterBytes), the rest unchanged
        const uint64_t tot = (uint64_t)(P.n + 2) * 8;
        const uint32_t total = (uint32_t)(tot < 0xFFFFFF00ull ? tot : 0xFFFFFF00ull);
        const uint32_t hot = (uint32_t)(P.hot_master_bytes < total ? P.hot_master_bytes : total);
        pol_keep = policy_masters(P.vs_t, hot, total);
    }
    extern __shared__ __align__(16) unsigned char dyn_smem[];
    __shared__ int s_done;
    Proxies px{nullptr, nullptr, 0};
    uint4* gbuf = nullptr;
    if (kAccum) {
        gbuf = reinterpret_cast<uint4*>(dyn_smem) + (size_t)(threadIdx.x >> 5) * kRing * 128;
        px.H = P.n_proxy;
        px.T = reinterpret_cast<unsigned long long*>(dyn_smem + gbuf_bytes<NW>());
        px.acc = reinterpret_cast<unsigned*>(px.T + px.H);
    }
    Acc acc;
    constexpr bool multi = MR;
    int r = 0, since = 0;
    unsigned long long ex = 0;
    __shared__ unsigned s_queue[2];
    for (; r < P.max_rounds; r++) {
        const int round = P.ctr->round + r;  // ctr->round only changes after the loop
        const int cur = round & 1, nxt = cur ^ 1;
        // this round's partition queues (per CTA, with stealing; or the global ticket)
        if (threadIdx.x == 0) { s_queue[0] = 1u; s_queue[1] = 0u; }
        __syncthreads();
        const Queue dq{P.qtick ? P.qtick + (size_t)cur * kQStride * gridDim.x : nullptr, &P.ctr->ticket[cur], s_queue};
        // a rank of a fused multi-rank run keeps going without local work: it
        // idles through rounds to the next exchange (mr_exchange)
        const bool idle = *((volatile unsigned*)&P.ctr->active[cur]) == 0;
        if (idle && !multi) break;
        const uint32_t* bcur = P.bits + (int64_t)cur * P.nw;
        uint32_t* bnxt = P.bits + (int64_t)nxt * P.nw;
        bool dense = !(multi && idle);  // this round streams every window (for the byte model)
        if (multi && idle) {
            if (kAccum)  // no sweep writes the next bitmap this round
                for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < P.nw;
                     i += (int64_t)gridDim.x * blockDim.x)
                    bnxt[i] = 0u;
        } else if constexpr (kAccum) {
            // sparse round: few signalled vertices whose out-edges are at most M / sparse_div
            if (sparse_round(P, grid, cur, bcur)) {
                dense = false;
                walk_sparse_acc<NW>(P, P.occ_items, *((volatile unsigned*)&P.ctr->qcur[cur]), &P.ctr->ticket[cur], bcur, acc);
            } else {
            if (EXP_ON(P, 96)) {  // DG_EXP 32: gather this round's start snapshot; 64: the previous round's
                unsigned long long* dst = P.snap + (size_t)((P.n + 3) & ~1ll) * (round & 1);
                if (blockIdx.x == 0 && threadIdx.x == 0) g_exp_par = EXP_ON(P, 32) ? (round & 1) : ((round + 1) & 1);
                for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < P.n + 2; i += (int64_t)gridDim.x * blockDim.x)
                    dst[i] = __ldcg(&P.vs_t[i]);
                grid.sync();
            }
            if (px.H) {  // round-start snapshot of the proxied masters
                for (int64_t i = threadIdx.x; i < px.H; i += blockDim.x) {
                    px.T[i] = __ldcg(&P.vs_t[i]);
                    px.acc[2 * i] = px.acc[2 * i + 1] = 0u;
                }
                if (threadIdx.x == 0) s_done = 0;
                __syncthreads();
            }
            walk_accum<ALGO == DG_ADSORPTION>(P, dq, acc, pol_stream, pol_keep, px, gbuf, &s_done);
            if (px.H) {  // send the proxies' accumulated pushes to their masters
                __syncthreads();
                for (int64_t i = threadIdx.x; i < px.H; i += blockDim.x)
                    if (const unsigned long long a = px_read(&px.acc[2 * i])) atomicAdd(&P.vs_t[i], a);
            }
            }
            grid.sync();  // all pushes of the round landed
            accum_sweep(P, bnxt, acc.sig);
        } else {
            unsigned* ticket = &P.ctr->ticket[cur];
            // bucket bound of this round (reading R-DELTA): only distances <= theta are committed
            const uint32_t theta = ((ALGO == DG_SSSP || ALGO == DG_BFS) && P.delta)
                                       ? sat_add(*(volatile unsigned*)&P.ctr->minval[cur], P.delta) : INF;
            // sparse round: when few vertices are
            // signalled, compact them; walk from them if their out-edges are
            // at most 1/sparse_div of the path entries, else walk the windows
            const bool sparse = (ALGO == DG_SSSP || ALGO == DG_BFS || ALGO == 100) && sparse_round(P, grid, cur, bcur);
            // probe-free dense round: most vertices signalled, or the signalled
            // ones own most out-edges (counted by sparse_round)
            const unsigned nact = *((volatile unsigned*)&P.ctr->active[cur]);
            const bool all = P.probe_free_occ &&
                             (nact > P.probe_free_act ||
                              (P.occ_off && (ALGO == DG_SSSP || ALGO == DG_BFS || ALGO == 100) &&
                               *((volatile unsigned*)&P.ctr->osum[cur]) >= P.probe_free_occ));
            if (sparse) {
                dense = false;
                const unsigned qn = *((volatile unsigned*)&P.ctr->qcur[cur]);
                if (ALGO == DG_SSSP) walk_sparse<0>(P, P.occ_off, P.occ, P.occ_items, qn, ticket, bnxt, theta, acc);
                else if (ALGO == DG_BFS) walk_sparse<1>(P, P.occ_off, P.occ, P.occ_items, qn, ticket, bnxt, theta, acc);
                else walk_sparse<3>(P, P.occ_off, P.occ, P.occ_items, qn, ticket, bnxt, theta, acc);
            } else if (ALGO == DG_SSSP) walk_minplus<0>(P, dq, bcur, bnxt, theta, acc, all);
            else if (ALGO == DG_BFS) walk_minplus<1>(P, dq, bcur, bnxt, theta, acc, all);
            else if (ALGO == DG_WCC) {
                // sparse WCC round: labels go forward along the out-edges, then
                // backward along the in-edges of the signalled vertices
                bool wsparse = false;
                if (P.occ_off && P.iocc_off && *((volatile unsigned*)&P.ctr->active[cur]) <= P.sparse_max) {
                    count_bits(P, P.occ_off, bcur, &P.ctr->qn[cur], &P.ctr->osum[cur]);
                    count_bits(P, P.iocc_off, bcur, &P.ctr->qn_in[cur], &P.ctr->osum_in[cur]);
                    grid.sync();
                    wsparse = (uint64_t)*((volatile unsigned*)&P.ctr->osum[cur]) +
                                  *((volatile unsigned*)&P.ctr->osum_in[cur]) <= P.sparse_occ;
                }
                if (wsparse) {
                    dense = false;
                    compact_bits(P, P.occ_off, bcur, P.occ_items, &P.ctr->qcur[cur]);
                    grid.sync();
                    walk_sparse<2>(P, P.occ_off, P.occ, P.occ_items, *((volatile unsigned*)&P.ctr->qn[cur]), ticket,
                                   bnxt, INF, acc);
                    grid.sync();  // the item buffer is reused
                    compact_bits(P, P.iocc_off, bcur, P.occ_items, &P.ctr->qcur_in[cur]);
                    grid.sync();
                    walk_sparse_bwd<true>(P, P.iocc_off, P.iocc, P.occ_items, *((volatile unsigned*)&P.ctr->qn_in[cur]),
                                          &P.ctr->ticket_in[cur], bnxt, acc);
                } else {
                    walk_minplus<2>(P, dq, bcur, bnxt, INF, acc, all);
                }
            }
            else if (ALGO == 100) walk_minplus<3>(P, dq, bcur, bnxt, INF, acc, all);
            else if (ALGO == 101 && sparse_round(P, grid, cur, bcur)) {
                // sparse backward round (same decision as the forward rounds)
                dense = false;
                walk_sparse_bwd<false>(P, P.occ_off, P.occ, P.occ_items, *((volatile unsigned*)&P.ctr->qcur[cur]), ticket, bnxt, acc);
            } else if (ALGO == 101) {
                while (true) {
                    const unsigned t = next_partition(P, dq);
                    if (t == kNoPart) break;
                    walk_scc_bwd(P, P.part_off[t], P.part_off[t + 1], bcur, bnxt, acc);
                }
            }
        }
        // publish this round's newly signalled vertices (the device active counter)
        unsigned s = acc.sig;
        for (int off = 16; off; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
        // a warp adds at most 2^19: with at most 148 x 4 x 8 warps the 32-bit
        // counter cannot wrap to 0 (it is an upper bound on the signalled
        // vertices, used only for its non-zero test and the sparse threshold)
        if (lane == 0 && s) atomicAdd(&P.ctr->active[nxt], min(s, 1u << 19));
        acc.sig = 0;
        if ((ALGO == DG_SSSP || ALGO == DG_BFS) && P.delta) {
            uint32_t mv = acc.vmin;
            for (int off = 16; off; off >>= 1) mv = min(mv, __shfl_xor_sync(0xffffffffu, mv, off));
            if (lane == 0 && mv != INF) atomicMin(&P.ctr->minval[nxt], mv);
            acc.vmin = INF;
        }
        grid.sync();
        if (P.qtick && threadIdx.x == 0) P.qtick[((size_t)cur * gridDim.x + blockIdx.x) * kQStride] = 0u;
        if (!kAccum) {  // retire this round's bitmap for reuse two rounds later
            uint32_t* bc = P.bits + (int64_t)cur * P.nw;
            for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < P.nw;
                 i += (int64_t)gridDim.x * blockDim.x)
                bc[i] = 0u;
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            if (P.trace && r < P.trace_cap) {  // developer trace (DG_TRACE)
                unsigned long long t;
                asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
                P.trace[4 * r] = t;
                P.trace[4 * r + 1] = P.ctr->active[cur];
                P.trace[4 * r + 2] = dense;
                P.trace[4 * r + 3] = P.ctr->osum[cur];
            }
            // a round whose pending relaxations were all beyond the bucket keeps the
            // bucket base; otherwise the next bucket starts at the smallest new distance
            if ((ALGO == DG_SSSP || ALGO == DG_BFS) && P.ctr->minval[nxt] == INF)
                P.ctr->minval[nxt] = sat_add(P.ctr->minval[cur], P.delta);
            P.ctr->active[cur] = 0;
            P.ctr->ticket[cur] = 0;
            P.ctr->minval[cur] = INF;
            if (dense) P.ctr->dense_rounds++;
            P.ctr->qn[cur] = 0;
            P.ctr->osum[cur] = 0;
            P.ctr->qcur[cur] = 0;
            P.ctr->qn_in[cur] = P.ctr->osum_in[cur] = P.ctr->qcur_in[cur] = P.ctr->ticket_in[cur] = 0;
        }
        grid.sync();
        if (multi && (++since >= P.mr.every || *((volatile unsigned*)&P.ctr->active[nxt]) == 0)) {
            since = 0;
            if (mr_exchange(P, grid, nxt, P.mr.epoch0 + ++ex)) {
                r++;
                break;
            }
        }
    }
    unsigned long long su = acc.upd, se = acc.edges, sn = acc.entries;
    for (int off = 16; off; off >>= 1) {
        su += __shfl_xor_sync(0xffffffffu, su, off);
        se += __shfl_xor_sync(0xffffffffu, se, off);
        sn += __shfl_xor_sync(0xffffffffu, sn, off);
    }
    if (lane == 0) {  // units are warp-uniform (counted identically by every lane)
        atomicAdd(&P.ctr->updates, su);
        atomicAdd(&P.ctr->edges, se);
        atomicAdd(&P.ctr->units, (unsigned long long)acc.units);
        atomicAdd(&P.ctr->entries, sn);
    }
    grid.sync();
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        P.ctr->round += r;
        P.ctr->mr_ex = ex;
        if (P.ctr_out) {  // the host reads the counters without a copy call after the launch
            const unsigned* src = reinterpret_cast<const unsigned*>(P.ctr);
            volatile unsigned* dst = reinterpret_cast<volatile unsigned*>(P.ctr_out);
            for (size_t k = 0; k < sizeof(Counters) / 4; k++) dst[k] = __ldcg(src + k);  // L2: other blocks' atomics
            __threadfence_system();
        }
    }
}

// ------------------------------------------------------------------ vertex-centric ablation
// Frontier kernel over the CSR (the synchronous vertex-centric model of the
// systems the paper compares against, sec. 2): every round each
// frontier vertex pushes along all its out-edges; warps load-balance the
// edges of 32 frontier vertices with a prefix sum.  "Updates" count writes to
// master states (successful relaxations; PageRank: delta pushes and folds).
template <int ALGO>
__global__ void __launch_bounds__(kBlock) vertex_kernel(KParams P) {
    cg::grid_group grid = cg::this_grid();
    __shared__ int64_t s_off[kWarps][33];
    __shared__ int32_t s_v[kWarps][32];
    __shared__ float s_push[kWarps][32];
    __shared__ uint32_t s_dist[kWarps][32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    Acc acc;
    int r = 0;
    for (; r < P.max_rounds; r++) {
        const int round = P.ctr->round + r;
        const int cur = round & 1, nxt = cur ^ 1;
        const unsigned ncur = *((volatile unsigned*)&P.ctr->active[cur]);
        if (ncur == 0) break;
        const int32_t* list = cur ? P.vlist1 : P.vlist0;
        int32_t* out = nxt ? P.vlist1 : P.vlist0;
        while (true) {
            unsigned t = 0;
            if (lane == 0) t = atomicAdd(&P.ctr->ticket[cur], 32u);
            t = __shfl_sync(0xffffffffu, t, 0);
            if (t >= ncur) break;
            int v = -1;
            int64_t deg = 0;
            if (t + lane < ncur) {
                v = list[t + lane];
                deg = P.row_ptr[v + 1] - P.row_ptr[v];
                acc.units++;
                if (ALGO == DG_PAGERANK) {
                    float4* s = &P.vs_f[v];
                    float d = atomicExch(&s->z, 0.f);
                    if (d > 0.f) { s->x += d; acc.upd++; }
                    s_push[wid][lane] = d * s->y;
                    if (!(d > 0.f)) deg = 0;
                } else {
                    s_dist[wid][lane] = P.vs_u[v];
                }
            }
            s_v[wid][lane] = v;
            int64_t inc = deg;
            for (int off = 1; off < 32; off <<= 1) {
                int64_t y = __shfl_up_sync(0xffffffffu, inc, off);
                if (lane >= off) inc += y;
            }
            s_off[wid][lane + 1] = inc;
            if (lane == 0) s_off[wid][0] = 0;
            __syncwarp();
            const int64_t total = s_off[wid][32];
            for (int64_t j = lane; j < total; j += 32) {
                int lo = 0, hi = 31;  // owner: largest o with s_off[o] <= j
                while (lo < hi) {
                    int mid = (lo + hi + 1) >> 1;
                    if (s_off[wid][mid] <= j) lo = mid; else hi = mid - 1;
                }
                const int u = s_v[wid][lo];
                const int64_t e = P.row_ptr[u] + (j - s_off[wid][lo]);
                const int x = P.col[e];
                acc.pushes++;
                bool push = false;
                if (ALGO == DG_PAGERANK) {
                    float a = s_push[wid][lo];
                    float old = atomicAdd(&P.vs_f[x].z, a);
                    acc.upd++;
                    push = old < P.eps && old + a >= P.eps;
                } else {
                    const uint32_t cand = ALGO == DG_WCC ? s_dist[wid][lo]
                                        : sat_add(s_dist[wid][lo], ALGO == DG_BFS ? 1u : (uint32_t)P.w[e]);
                    if (cand < P.vs_u[x]) {
                        uint32_t old = atomicMin(&P.vs_u[x], cand);
                        if (cand < old) { acc.upd++; push = true; }
                    }
                }
                if (push) {
                    unsigned* stp = ALGO == DG_PAGERANK ? reinterpret_cast<unsigned*>(&P.vs_f[x].w) : &P.vstamp[x];
                    if (atomicExch(stp, (unsigned)(round + 1)) != (unsigned)(round + 1)) {
                        unsigned slot = atomicAdd(&P.ctr->active[nxt], 1u);
                        out[slot] = x;
                    }
                }
            }
            __syncwarp();
        }
        grid.sync();
        if (blockIdx.x == 0 && threadIdx.x == 0) { P.ctr->active[cur] = 0; P.ctr->ticket[cur] = 0; }
        grid.sync();
    }
    unsigned long long su = acc.upd, sn = acc.units, sp = acc.pushes;
    for (int off = 16; off; off >>= 1) {
        su += __shfl_xor_sync(0xffffffffu, su, off);
        sn += __shfl_xor_sync(0xffffffffu, sn, off);
        sp += __shfl_xor_sync(0xffffffffu, sp, off);
    }
    if (lane == 0) {
        atomicAdd(&P.ctr->updates, su);
        atomicAdd(&P.ctr->edges, sp);
        atomicAdd(&P.ctr->units, sn);
        atomicAdd(&P.ctr->pushes, sp);
    }
    grid.sync();
    if (blockIdx.x == 0 && threadIdx.x == 0) P.ctr->round += r;
}

// ------------------------------------------------------------------ small kernels
#define GRID_STRIDE(i, n) \
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (n); i += (int64_t)gridDim.x * blockDim.x)

// WCC labels start as the ORIGINAL vertex id (reading R-CC: smallest original id wins)
__global__ void init_u_kernel(uint32_t* vs, uint32_t* stamp, const int32_t* orig, int64_t n, int algo,
                              int64_t source) {
    GRID_STRIDE(v, n) {
        vs[v] = (algo == DG_WCC) ? (uint32_t)orig[v] : (v == source ? 0u : INF);
        stamp[v] = 0u;
    }
}
// SSSP sparse walks: each path entry's code and the weight of the path edge
// into it side by side, so a walk step is one random 8-byte load
__global__ void cw_build_kernel(uint2* cw, const uint32_t* e_idx, const int32_t* e_w, int64_t n) {
    GRID_STRIDE(i, n) cw[i] = make_uint2(e_idx[i], (uint32_t)e_w[i]);
}
// path-mode SSSP/BFS start state in one launch: distances (source 0),
// bitmaps zeroed except the source's bit in bitmap 0, the run's counters
__global__ void init_minplus_kernel(uint32_t* vs, uint32_t* stamp, int64_t n, int64_t source, uint32_t* bits,
                                    int64_t nbits_words, Counters* ctr, Counters c) {
    const int64_t T = (int64_t)gridDim.x * blockDim.x;
    const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (int64_t v = t0; v < n; v += T) {
        vs[v] = v == source ? 0u : INF;
        stamp[v] = 0u;
    }
    for (int64_t i = t0; i < nbits_words; i += T) bits[i] = i == (source >> 5) ? 1u << (source & 31) : 0u;
    if (t0 == 0) *ctr = c;
}
// vertex-centric ablation: {r, g, delta, stamp} = {0, d/outdeg, 1-d, 0}
// (unnormalised delta PageRank, reading R-PR)
__global__ void init_pr_kernel(float4* vs, const int32_t* outdeg, int64_t n, float d) {
    GRID_STRIDE(v, n) {
        float c = outdeg[v] > 0 ? d / (float)outdeg[v] : 0.f;
        vs[v] = make_float4(0.f, c, 1.f - d, 0.f);
    }
}
// path mode: T = 1-d (PageRank) or p_inj*I (Adsorption, base != null), sigma = T
__global__ void init_acc_kernel(unsigned long long* vs, unsigned long long* sigma, const float* base, int64_t n,
                                float d) {
    GRID_STRIDE(v, n) {
        const float t0 = base ? base[v] : 1.f - d;
        const unsigned long long T = (unsigned long long)((double)t0 * 4294967296.0);
        vs[v] = T;  // S_val = 0: every entry has pend = T >= eps in round 0
        sigma[v] = T;
    }
}
// PageRank: coefficient of the path edge out of entry i = d / outdeg(v_i)
__global__ void pr_coef_kernel(float* e_coef, const uint32_t* e_idx, const int32_t* outdeg, float d, int64_t M) {
    GRID_STRIDE(i, M) {
        const uint32_t c = e_idx[i];
        const int32_t od = outdeg[c & kVMask];
        e_coef[i] = (!(c & kTail) && od > 0) ? d / (float)od : 0.f;
    }
}
__global__ void fill_iota_kernel(int32_t* a, int64_t n) {
    GRID_STRIDE(i, n) a[i] = (int32_t)i;
}
// all vertices signalled (bits 0..n-1 set, the rest clear)
__global__ void bits_all_kernel(uint32_t* b, int64_t nw, int64_t n) {
    GRID_STRIDE(i, nw) {
        const int64_t lo = i * 32;
        b[i] = (n - lo >= 32) ? 0xffffffffu : (n > lo ? ((1u << (n - lo)) - 1u) : 0u);
    }
}
__global__ void bits_set_one_kernel(uint32_t* b, int64_t v) { b[v >> 5] |= 1u << (v & 31); }
// Adsorption: coefficient of the path edge out of entry i = p_cont(u) * w(u, next) / W(u)
__global__ void ads_coef_kernel(float* e_coef, const uint32_t* e_idx, const int32_t* e_w, const float* pcont,
                                const float* wsum, int64_t M) {
    GRID_STRIDE(i, M) {
        uint32_t c = e_idx[i];
        float x = 0.f;
        if (!(c & kTail)) {
            uint32_t u = c & kVMask;
            x = pcont[u] * (float)e_w[i + 1] / wsum[u];
        }
        e_coef[i] = x;
    }
}
__device__ __forceinline__ double final_value(const float4* vf, const unsigned long long* va, int64_t v) {
    if (va) return (double)va[v] * (1.0 / 4294967296.0);
    float4 x = vf[v];
    return (double)x.x + (double)x.z;  // ablation: r + pending delta
}
__global__ void sum_T_kernel(const float4* vf, const unsigned long long* va, int64_t n, double* out) {
    double s = 0;
    GRID_STRIDE(v, n) s += final_value(vf, va, v);
    for (int off = 16; off; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    if ((threadIdx.x & 31) == 0) atomicAdd(out, s);
}
// outputs are indexed by ORIGINAL vertex id: out[v] = state[new_id[v]]
__global__ void out_pr_kernel(const float4* vf, const unsigned long long* va, const int32_t* new_id, int64_t n,
                              const double* sum, float* out, int normalize) {
    const double inv = normalize ? 1.0 / *sum : 1.0;
    GRID_STRIDE(v, n) out[v] = (float)(final_value(vf, va, new_id[v]) * inv);
}
__global__ void out_u_kernel(const uint32_t* vs, const int32_t* new_id, int64_t n, uint32_t* out) {
    GRID_STRIDE(v, n) out[v] = vs[new_id[v]];
}
__global__ void out_i_kernel(const int32_t* x, const int32_t* new_id, int64_t n, int32_t* out) {
    GRID_STRIDE(v, n) out[v] = x[new_id[v]];
}
__global__ void sum_f_kernel(const float* x, int64_t n, double* out) {
    double s = 0;
    GRID_STRIDE(v, n) s += (double)x[v];
    for (int off = 16; off; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    if ((threadIdx.x & 31) == 0) atomicAdd(out, s);
}
__global__ void scale_f_kernel(float* x, int64_t n, const double* sum) {
    const double inv = 1.0 / *sum;
    GRID_STRIDE(v, n) x[v] = (float)((double)x[v] * inv);
}

// ---- occurrence index (sparse min-plus rounds): vertex -> its non-tail entries
// (skip = kTail: out-edges, the entries a path edge leaves; skip = kHead:
// in-edges, the entries a path edge enters)
// Each block takes one contiguous chunk of entries.  The kOccHubs
// highest-degree vertices (internal ids [0, kOccHubs)) are counted in shared
// memory: their occurrences would otherwise serialise on a few global
// counters (R-MAT hubs hold hundreds of thousands of entries).
constexpr uint32_t kOccHubs = 4096;
constexpr int kOccBlocksPerSM = 8;
__device__ __forceinline__ void occ_chunk(int64_t M, int64_t& beg, int64_t& end) {
    const int64_t chunk = (M + gridDim.x - 1) / gridDim.x;
    beg = (int64_t)blockIdx.x * chunk;
    end = beg + chunk < M ? beg + chunk : M;
}
__global__ void __launch_bounds__(256) occ_count_kernel(const uint32_t* e_idx, int64_t M, uint32_t skip,
                                                        uint32_t hubs, uint32_t* cnt) {
    __shared__ uint32_t s[kOccHubs];
    for (uint32_t h = threadIdx.x; h < hubs; h += blockDim.x) s[h] = 0;
    __syncthreads();
    int64_t beg, end;
    occ_chunk(M, beg, end);
    for (int64_t i = beg + threadIdx.x; i < end; i += blockDim.x) {
        const uint32_t c = __ldcs(e_idx + i);
        if (c & skip) continue;
        const uint32_t v = c & kVMask;
        if (v < hubs) atomicAdd(&s[v], 1u);
        else atomicAdd(&cnt[v + 1], 1u);
    }
    __syncthreads();
    for (uint32_t h = threadIdx.x; h < hubs; h += blockDim.x)
        if (s[h]) atomicAdd(&cnt[h + 1], s[h]);
}
// Same chunks: the block recounts its hub occurrences, reserves one range per
// hub with a single global atomic, then places every occurrence (hubs from
// their shared-memory cursor, the others from the global one).
__global__ void __launch_bounds__(256) occ_fill_kernel(const uint32_t* e_idx, int64_t M, uint32_t skip,
                                                       uint32_t hubs, uint32_t* cursor, uint32_t* occ) {
    __shared__ uint32_t s[kOccHubs];
    for (uint32_t h = threadIdx.x; h < hubs; h += blockDim.x) s[h] = 0;
    __syncthreads();
    int64_t beg, end;
    occ_chunk(M, beg, end);
    for (int64_t i = beg + threadIdx.x; i < end; i += blockDim.x) {
        const uint32_t c = e_idx[i];
        if (!(c & skip) && (c & kVMask) < hubs) atomicAdd(&s[c & kVMask], 1u);
    }
    __syncthreads();
    for (uint32_t h = threadIdx.x; h < hubs; h += blockDim.x)
        if (s[h]) s[h] = atomicAdd(&cursor[h], s[h]);
    __syncthreads();
    // four entries per thread and step: their atomics are in flight together
    constexpr int kU = 4;
    for (int64_t i0 = beg + (int64_t)threadIdx.x * kU; i0 < end; i0 += (int64_t)blockDim.x * kU) {
        uint32_t c[kU], pos[kU];
#pragma unroll
        for (int u = 0; u < kU; u++) c[u] = i0 + u < end ? __ldcs(e_idx + i0 + u) : skip;
#pragma unroll
        for (int u = 0; u < kU; u++) {
            const uint32_t v = c[u] & kVMask;
            pos[u] = (c[u] & skip) ? 0u : (v < hubs ? atomicAdd(&s[v], 1u) : atomicAdd(&cursor[v], 1u));
        }
#pragma unroll
        for (int u = 0; u < kU; u++)
            if (!(c[u] & skip)) occ[pos[u]] = (uint32_t)(i0 + u);
    }
}

// ---- SCC helpers
// colours are ORIGINAL vertex ids so an SCC's label is its smallest original id
__global__ void scc_init_kernel(uint32_t* vs, const int32_t* label, const int32_t* orig, uint8_t* mark, int64_t n) {
    GRID_STRIDE(v, n) {
        vs[v] = label[v] < 0 ? (uint32_t)orig[v] : INF;
        mark[v] = 0;
    }
}
// the forward phase starts with every unassigned vertex signalled
__global__ void scc_bits_kernel(const int32_t* label, int64_t n, uint32_t* b, int64_t nw) {
    GRID_STRIDE(i, nw) {
        uint32_t w = 0;
        for (int k = 0; k < 32; k++) {
            const int64_t v = i * 32 + k;
            if (v < n && label[v] < 0) w |= 1u << k;
        }
        b[i] = w;
    }
}
// roots keep their own id as colour; they seed the backward phase's bitmap
__global__ void scc_roots_kernel(const uint32_t* vs, const int32_t* label, const int32_t* orig, uint8_t* mark,
                                 int64_t n, uint32_t* b, Counters* ctr) {
    unsigned cnt = 0;
    GRID_STRIDE(v, n) {
        const bool root = label[v] < 0 && vs[v] == (uint32_t)orig[v];
        mark[v] = root;
        if (root) cnt += signal_vertex(b, (uint32_t)v);
    }
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(&ctr->active[0], cnt);
}
__global__ void scc_assign_kernel(const uint32_t* vs, int32_t* label, const uint8_t* mark, int64_t n, int32_t* remaining) {
    int cnt = 0;
    GRID_STRIDE(v, n) {
        if (label[v] < 0) {
            if (mark[v]) label[v] = (int32_t)vs[v];
            else cnt++;
        }
    }
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(remaining, cnt);
}

// ---- multi-GPU boundary exchange ("each mirror always
// sends its new state to its master"; line 96: synchronisation in batches)
// MIN exchanges; with `mark` set (SCC backward phase) the replicated state is
// the reachability mark, encoded 0 = marked / 1 = not, so MIN is OR.
__device__ __forceinline__ uint32_t min_value(const uint32_t* vs, const uint8_t* mark, int v) {
    return mark ? (mark[v] ? 0u : 1u) : vs[v];
}
__device__ __forceinline__ bool min_apply(uint32_t* vs, uint8_t* mark, const int32_t* label, int v, uint32_t m) {
    if (mark) {
        if (m != 0u || mark[v] || label[v] >= 0) return false;
        mark[v] = 1;
        return true;
    }
    if (m >= vs[v]) return false;
    vs[v] = m;
    return true;
}
__global__ void pack_min_kernel(const uint32_t* vs, const uint8_t* mark, const int32_t* bnd, int64_t nb, uint32_t* buf) {
    GRID_STRIDE(k, nb) buf[k] = min_value(vs, mark, bnd[k]);
}
__global__ void unpack_min_kernel(uint32_t* vs, uint8_t* mark, const int32_t* label, const int32_t* bnd, int64_t nb,
                                  const uint32_t* buf, uint32_t* b, Counters* ctr, int slot) {
    unsigned cnt = 0;
    GRID_STRIDE(k, nb) {
        const int v = bnd[k];
        if (min_apply(vs, mark, label, v, buf[k])) cnt += signal_vertex(b, (uint32_t)v);
    }
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(&ctr->active[slot], cnt);
}
// SUM algorithms exchange the growth of each boundary total since the last
// exchange; after the all-reduce every replica holds the same total.
__global__ void init_base_kernel(const unsigned long long* vs, const int32_t* bnd, int64_t nb, unsigned long long* base) {
    GRID_STRIDE(k, nb) base[k] = vs[bnd[k]];
}
__global__ void pack_sum_kernel(const unsigned long long* vs, const int32_t* bnd, int64_t nb,
                                const unsigned long long* base, unsigned long long* buf) {
    GRID_STRIDE(k, nb) buf[k] = vs[bnd[k]] - base[k];
}
__global__ void unpack_sum_kernel(unsigned long long* vs, unsigned long long* sigma, const int32_t* bnd, int64_t nb,
                                  unsigned long long* base, const unsigned long long* buf, unsigned long long eps,
                                  uint32_t* b, Counters* ctr, int slot) {
    unsigned cnt = 0;
    GRID_STRIDE(k, nb) {
        const int v = bnd[k];
        const unsigned long long t = base[k] + buf[k];
        base[k] = t;
        vs[v] = t;
        if (t - sigma[v] >= eps) {  // the replica's growth counts as a signal of the next local round
            sigma[v] = t;
            signal_vertex(b, (uint32_t)v);  // (the bitmap sparse rounds read)
            cnt++;
        }
    }
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(&ctr->active[slot], cnt);
}

// ---- peer-memory boundary exchange (replaces pack + NCCL all-reduce + unpack)
// Every rank owns one exchange region in its HBM, mapped into every peer by
// CUDA IPC (NVLink/NVSwitch loads and stores between B200s):
//   [flags: kP2PMaxRanks x u64 epochs written by the peers | error word]
//   [slot 0: n_bnd x u64][slot 1: n_bnd x u64]      (double buffer by epoch parity)
// Exchange e: (1) pack this rank's boundary values into its own slot e&1;
// (2) one warp publishes epoch e into every peer's flag word for this rank
// (release, system scope) and waits until every peer published e here
// (acquire); (3) every rank reduces all ranks' slot e&1 elementwise (MIN, or
// SUM of growth) straight from peer memory and applies it like unpack.  A
// rank rewrites slot e&1 only at exchange e+2, after every peer published
// e+1, i.e. after every peer's exchange-e reduce completed (stream order).
struct PeerSlots {
    const void* p[kP2PMaxRanks];
};
__global__ void p2p_pack_min_kernel(const uint32_t* vs, const uint8_t* mark, const int32_t* bnd,
                                    const unsigned long long* hold, int rank, int64_t nb, unsigned long long* slot) {
    GRID_STRIDE(k, nb) if ((hold[k] >> rank) & 1ull) slot[k] = min_value(vs, mark, bnd[k]);
}
__global__ void p2p_pack_sum_kernel(const unsigned long long* vs, const int32_t* bnd, const unsigned long long* hold,
                                    int rank, int64_t nb, const unsigned long long* base, unsigned long long* slot) {
    GRID_STRIDE(k, nb) if ((hold[k] >> rank) & 1ull) slot[k] = vs[bnd[k]] - base[k];
}
__global__ void p2p_signal_wait_kernel(PeerSlots flags, int world, int rank, unsigned long long epoch,
                                       unsigned long long* own_flags, unsigned long long timeout_ns) {
    const int q = threadIdx.x;
    if (q < world && q != rank) {
        __threadfence_system();
        unsigned long long* f = (unsigned long long*)flags.p[q] + rank;
        asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(epoch) : "memory");
    }
    __syncwarp();
    if (q < world && q != rank) {
        unsigned long long t0, t, v;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
        while (true) {
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(own_flags + q) : "memory");
            if (v >= epoch) break;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            if (t - t0 > timeout_ns) {  // a peer never arrived: report instead of hanging the GPU
                atomicExch(own_flags + kP2PErr, 1ull);
                break;
            }
            __nanosleep(256);
        }
    }
}
__global__ void p2p_reduce_min_kernel(PeerSlots slots, int rank, uint32_t* vs, uint8_t* mark, const int32_t* label,
                                      const int32_t* bnd, const unsigned long long* hold, int64_t nb, uint32_t* b,
                                      Counters* ctr, int slot) {
    unsigned cnt = 0;
    GRID_STRIDE(k, nb) {
        const unsigned long long hm = hold[k];
        if (!((hm >> rank) & 1ull)) continue;
        unsigned long long m = ~0ull;
        for (unsigned long long q = hm; q; q &= q - 1)
            m = min(m, __ldcv((const unsigned long long*)slots.p[__ffsll((long long)q) - 1] + k));
        const int v = bnd[k];
        if (min_apply(vs, mark, label, v, (uint32_t)m)) cnt += signal_vertex(b, (uint32_t)v);
    }
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(&ctr->active[slot], cnt);
}
__global__ void p2p_reduce_sum_kernel(PeerSlots slots, int rank, unsigned long long* vs, unsigned long long* sigma,
                                      const int32_t* bnd, const unsigned long long* hold, int64_t nb,
                                      unsigned long long* base, unsigned long long eps, uint32_t* b, Counters* ctr,
                                      int slot) {
    unsigned cnt = 0;
    GRID_STRIDE(k, nb) {
        const unsigned long long hm = hold[k];
        if (!((hm >> rank) & 1ull)) continue;
        unsigned long long g = 0;
        for (unsigned long long q = hm; q; q &= q - 1)
            g += __ldcv((const unsigned long long*)slots.p[__ffsll((long long)q) - 1] + k);
        const int v = bnd[k];
        const unsigned long long t = base[k] + g;
        base[k] = t;
        vs[v] = t;
        if (t - sigma[v] >= eps) {
            sigma[v] = t;
            signal_vertex(b, (uint32_t)v);
            cnt++;
        }
    }
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(&ctr->active[slot], cnt);
}

// ------------------------------------------------------------------ host side
namespace {

template <typename T>
int dalloc(T** p, size_t count, int64_t& bytes, std::string& err) {
    size_t b = sizeof(T) * (count ? count : 1);
    cudaError_t e = cudaMalloc((void**)p, b);
    if (e != cudaSuccess) {
        err = std::string("cudaMalloc(") + std::to_string(b) + "): " + cudaGetErrorString(e);
        return e == cudaErrorMemoryAllocation ? DG_ENOMEM : DG_ENOCUDA;
    }
    bytes += (int64_t)b;
    return DG_OK;
}
template <typename T>
int dalloc_once(T** p, size_t count, int64_t& bytes, std::string& err) {
    return *p ? DG_OK : dalloc(p, count, bytes, err);
}
template <typename T>
void dfree(T*& p) {
    if (p) cudaFree((void*)p);
    p = nullptr;
}
int64_t* g_h2d_counter = nullptr;           // DevLayout::h2d_bytes of the upload in progress
std::vector<void*>* g_pin_list = nullptr;   // DevLayout::pinned of the upload in progress
template <typename T>
int h2d(T* dst, const T* src, size_t count, std::string& err) {
    if (!count) return DG_OK;
    // page-lock large host arrays once so uploads run at full link speed
    if (g_pin_list && sizeof(T) * count >= (1u << 20)) {
        void* hp = const_cast<T*>(src);
        bool have = false;
        for (void* q : *g_pin_list) have |= (q == hp);
        if (!have && cudaHostRegister(hp, sizeof(T) * count, cudaHostRegisterPortable) == cudaSuccess)
            g_pin_list->push_back(hp);
        cudaGetLastError();
    }
    CK(cudaMemcpy(dst, src, sizeof(T) * count, cudaMemcpyHostToDevice));
    if (g_h2d_counter) *g_h2d_counter += (int64_t)(sizeof(T) * count);
    return DG_OK;
}
int grid_1d(int64_t n) {
    int64_t g = (n + 255) / 256;
    return (int)std::max<int64_t>(1, std::min<int64_t>(g, 148 * 16));
}

KParams make_params(const DevLayout& D, DevWork* W) {
    KParams P{};
    P.e_idx = D.e_idx; P.e_w = D.e_w; P.part_off = D.part_off;
    P.row_ptr = D.row_ptr; P.col = D.col; P.w = D.w;
    P.n_part = D.n_part; P.n = D.n; P.nw = W->nw;
    P.vs_u = W->vs_u; P.vstamp = W->vstamp; P.vs_f = W->vs_f; P.vs_t = W->vs_t; P.sigma = W->sigma; P.s_val = W->s_val;
    P.e_coef = W->e_coef; P.bits = W->bits;
    P.vlist0 = W->vlist[0]; P.vlist1 = W->vlist[1];
    P.ctr = W->ctr;
    P.mark = W->scc_mark; P.scc_label = W->scc_label;
    P.orig = D.orig; P.n_proxy = D.n_proxy;
    // partition dispatch: one global ticket in priority order (default), or
    // per-CTA queues with work stealing (DG_DISPATCH=1, developer knob;
    // measured slower, DESIGN.md sec. 4 "Dispatch")
    const char* dd = std::getenv("DG_DISPATCH");
    P.qtick = (dd && std::atoi(dd) == 1) ? W->qtick : nullptr;
    return P;
}

int ensure_work(DevWork*& W, const DevLayout& D, std::string& err) {
    if (W) return DG_OK;
    W = new DevWork();
    int64_t bytes = 0;
    int rc;
    W->nw = (D.n + 31) / 32 + 1;
    if ((rc = dalloc(&W->vs_u, D.n + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->vstamp, D.n + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->vs_f, D.n + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->vs_t, D.n + 2, bytes, err))) return rc;
    if ((rc = dalloc(&W->sigma, D.n + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->s_val, D.M + kPad, bytes, err))) return rc;
    if ((rc = dalloc(&W->bnd_base, D.n_bnd + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->bits, 2 * W->nw, bytes, err))) return rc;
    if ((rc = dalloc(&W->vlist[0], D.n + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->vlist[1], D.n + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->ctr, 1, bytes, err))) return rc;
    if (cudaHostAlloc(&W->ctr_host, sizeof(Counters), cudaHostAllocMapped) != cudaSuccess ||
        cudaHostGetDevicePointer(&W->ctr_host_dev, W->ctr_host, 0) != cudaSuccess) {
        if (W->ctr_host) cudaFreeHost(W->ctr_host);
        W->ctr_host = W->ctr_host_dev = nullptr;  // optional: counters are then copied back
        cudaGetLastError();
    }
    if ((rc = dalloc(&W->dsum, 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->qtick, 2 * kMaxGrid * kQStride, bytes, err))) return rc;
    CK(cudaMemset(W->s_val, 0, sizeof(unsigned long long) * (D.M + kPad)));
    CK(cudaEventCreate(&W->ev0));
    CK(cudaEventCreate(&W->ev1));
    CK(cudaEventCreate(&W->kev0));
    CK(cudaEventCreate(&W->kev1));
    return DG_OK;
}

int read_counters(DevWork* W, Counters& c, std::string& err) {
    CK(cudaMemcpy(&c, W->ctr, sizeof(Counters), cudaMemcpyDeviceToHost));
    return DG_OK;
}
// the counters are set by a one-thread kernel in stream order (the struct
// travels as a kernel argument): no host synchronisation before the launch
__global__ void set_counters_kernel(Counters* ctr, Counters c) { *ctr = c; }
int write_counters(DevWork* W, const Counters& c, std::string& err, RunState* S = nullptr) {
    set_counters_kernel<<<1, 1>>>(W->ctr, c);
    CK(cudaGetLastError());
    if (S) S->stats.kernel_launches++;
    return DG_OK;
}

int coop_launch(DevWork* W, void* fn, KParams& P, RunState& S, std::string& err, size_t smem = 0,
                int threads = kBlock, int max_per_sm = 0) {
    // grid size per (device, kernel, block, shared memory), queried once:
    // the occupancy query and the attribute call cost tens of microseconds,
    // which small graphs (configs[0]: ~0.3 ms per run) would pay every run
    // (the dynamic shared-memory attribute is per kernel: it is set again
    // whenever a launch of that kernel asks for a different size)
    static std::mutex mu;
    static std::map<std::tuple<int, void*, int, size_t>, int> grids;
    static std::map<std::pair<int, void*>, size_t> smem_attr;
    int dev = 0;
    CK(cudaGetDevice(&dev));
    int grid = 0;
    {
        std::lock_guard<std::mutex> lk(mu);
        if (smem) {
            auto a = smem_attr.find({dev, fn});
            if (a == smem_attr.end() || a->second != smem) {
                CK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
                smem_attr[{dev, fn}] = smem;
            }
        }
        const auto key = std::make_tuple(dev, fn, threads, smem);
        auto it = grids.find(key);
        if (it == grids.end()) {
            int sms = 0, per = 0;
            CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
            CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, threads, smem));
            it = grids.emplace(key, std::min(sms * std::max(1, per), kMaxGrid)).first;
        }
        grid = it->second;
        if (max_per_sm > 0) {  // fewer resident CTAs than the occupancy allows (small graphs)
            int sms = 0;
            CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
            grid = std::min(grid, sms * max_per_sm);
        }
    }
    if (P.qtick) CK(cudaMemsetAsync(P.qtick, 0, sizeof(unsigned) * 2 * kMaxGrid * kQStride));
    void* args[] = {&P};
    CK(cudaEventRecord(W->kev0));
    CK(cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(threads), args, smem, 0));
    CK(cudaGetLastError());
    CK(cudaEventRecord(W->kev1));
    S.stats.kernel_launches++;
    if (W->defer_kernel_time) {  // dg_run: read after its own end event (one host wait per run)
        W->kernel_time_pending = true;
        return DG_OK;
    }
    CK(cudaEventSynchronize(W->kev1));
    float kms = 0;
    CK(cudaEventElapsedTime(&kms, W->kev0, W->kev1));
    S.stats.kernel_ms += kms;
    return DG_OK;
}


// Sparse min-plus rounds: a round with at most
// n/4 signalled vertices whose out-edges are at most M / DG_SPARSE_DIV walks
// from them; 0 disables.
int64_t sparse_div() {
    const char* e = std::getenv("DG_SPARSE_DIV");  // developer knob
    return e ? std::atoll(e) : 16;
}
// Below this many path entries a dense round costs less than a sparse round's
// two extra grid barriers and its dependent walk steps (measured: 1.1 M
// entries lose, 56 M and 73 M win).
int64_t sparse_min_entries() {
    const char* e = std::getenv("DG_SPARSE_MIN_M");  // developer knob
    return e ? std::atoll(e) : (int64_t)1 << 23;
}

// Occurrence index: counting sort of the non-tail (out-edge) or non-head
// (in-edge, SCC backward) entries by vertex, built on the device on the first
// run that needs it after an upload.
// Scratch (cursor, cub temporary) and the index arrays stay allocated across
// re-uploads of a layout of the same size; only the contents are rebuilt.
int build_occ(DevWork* W, const DevLayout& D, uint32_t skip, uint32_t*& off, uint32_t*& occ, int64_t& cap,
              RunState& S, std::string& err) {
    int64_t bytes = 0;
    int rc;
    const bool verbose = std::getenv("DG_VERBOSE") != nullptr;
    if (verbose) CK(cudaEventRecord(W->ev0));
    if (!off && (rc = dalloc(&off, D.n + 1, bytes, err))) return rc;
    if (!W->occ_cur && (rc = dalloc(&W->occ_cur, D.n + 1, bytes, err))) return rc;
    CK(cudaMemsetAsync(off, 0, sizeof(uint32_t) * (D.n + 1)));
    int dev = 0, sms = 148;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    const int oblocks = (int)std::max<int64_t>(1, std::min<int64_t>((int64_t)sms * kOccBlocksPerSM, (D.M + 255) / 256));
    const uint32_t hubs = (uint32_t)std::min<int64_t>(D.n, kOccHubs);
    occ_count_kernel<<<oblocks, 256>>>(D.e_idx, D.M, skip, hubs, off);
    size_t tmp_bytes = 0;
    CK(cub::DeviceScan::InclusiveSum(nullptr, tmp_bytes, off, off, (int)(D.n + 1)));
    if (tmp_bytes > W->cub_tmp_bytes) {
        if (W->cub_tmp) cudaFree(W->cub_tmp);
        CK(cudaMalloc(&W->cub_tmp, tmp_bytes));
        W->cub_tmp_bytes = tmp_bytes;
    }
    CK(cub::DeviceScan::InclusiveSum(W->cub_tmp, tmp_bytes, off, off, (int)(D.n + 1)));
    // capacity M + 1 bounds the occurrences (every path has a head and a
    // tail), so the build needs no device->host round trip
    if (D.M + 1 > cap) {
        dfree(occ);
        if ((rc = dalloc(&occ, (size_t)D.M + 1, bytes, err))) return rc;
        cap = D.M + 1;
    }
    CK(cudaMemcpyAsync(W->occ_cur, off, sizeof(uint32_t) * D.n, cudaMemcpyDeviceToDevice));
    occ_fill_kernel<<<oblocks, 256>>>(D.e_idx, D.M, skip, hubs, W->occ_cur, occ);
    CK(cudaGetLastError());
    S.stats.kernel_launches += 3;
    if (verbose) {
        CK(cudaEventRecord(W->ev1));
        CK(cudaEventSynchronize(W->ev1));
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, W->ev0, W->ev1));
        uint32_t total = 0;
        CK(cudaMemcpy(&total, off + D.n, sizeof(uint32_t), cudaMemcpyDeviceToHost));
        fprintf(stderr, "[dg] occurrence index (%s): %u entries in %.2f ms\n", skip == kTail ? "out" : "in", total, ms);
    }
    return DG_OK;
}
int ensure_occ(DevWork* W, const DevLayout& D, RunState& S, bool incoming, std::string& err) {
    int rc;
    if (!W->occ_items) {  // every path edge is one out- and one in-occurrence: one item buffer serves both
        int64_t bytes = 0;
        if ((rc = dalloc(&W->occ_items, (size_t)(D.n + D.m / kOccChunk + 1), bytes, err))) return rc;
    }
    if (incoming) {
        if (!W->iocc_ok && (rc = build_occ(W, D, kHead, W->iocc_off, W->iocc, W->iocc_cap, S, err))) return rc;
        W->iocc_ok = true;
    } else {
        if (!W->occ_ok && (rc = build_occ(W, D, kTail, W->occ_off, W->occ, W->occ_cap, S, err))) return rc;
        W->occ_ok = true;
    }
    return DG_OK;
}

// Launch the persistent path kernel for at most `rounds` rounds.
int launch_path(DevWork* W, const DevLayout& D, int algo_k, int rounds, RunState& S, std::string& err,
                const MultiRank* mr = nullptr) {
    KParams P = make_params(D, W);
    if (mr) P.mr = *mr;
    P.eps = (float)S.eps;
    P.eps_fx = (unsigned long long)(S.eps * 4294967296.0);
    P.max_rounds = rounds;
    void* fn = nullptr;
    if (mr) {
        switch (algo_k) {
            case DG_SSSP: fn = (void*)path_kernel<DG_SSSP, DG_PATH_MINB, true>; break;
            case DG_BFS: fn = (void*)path_kernel<DG_BFS, DG_PATH_MINB, true>; break;
            case DG_WCC: fn = (void*)path_kernel<DG_WCC, DG_PATH_MINB, true>; break;
            case DG_PAGERANK: fn = (void*)path_kernel<DG_PAGERANK, 1, true>; break;
            case DG_ADSORPTION: fn = (void*)path_kernel<DG_ADSORPTION, 1, true>; break;
            case 100: fn = (void*)path_kernel<100, DG_PATH_MINB, true>; break;
            case 101: fn = (void*)path_kernel<101, DG_PATH_MINB, true>; break;
            default: err = "fused multi-rank run: bad algo"; return DG_EINVAL;
        }
    } else switch (algo_k) {
        case DG_SSSP: fn = (void*)path_kernel<DG_SSSP>; break;
        case DG_BFS: fn = (void*)path_kernel<DG_BFS>; break;
        case DG_WCC: fn = (void*)path_kernel<DG_WCC>; break;
        case DG_PAGERANK: fn = (void*)path_kernel<DG_PAGERANK, 1>; break;
        case DG_ADSORPTION: fn = (void*)path_kernel<DG_ADSORPTION, 1>; break;
        case 100: fn = (void*)path_kernel<100>; break;
        case 101: fn = (void*)path_kernel<101>; break;
        default: err = "bad algo"; return DG_EINVAL;
    }
    const bool accum = algo_k == DG_PAGERANK || algo_k == DG_ADSORPTION;
    // ids are degree-descending, so any H' <= the built n_proxy also names
    // the H' highest-degree vertices: DG_N_PROXY caps the proxies per launch
    // (developer knob)
    if (const char* np = std::getenv("DG_N_PROXY")) P.n_proxy = std::min<int64_t>(P.n_proxy, std::max(0, std::atoi(np)));
    if (!accum) P.n_proxy = 0;
    {
        // refresh interval: about 16 mid-round flushes per CTA and round, at
        // least every 8 and at most every 128 partitions (measured: LJ-shaped
        // prefers 8-16, Twitter-shaped 64-128; DESIGN.md sec. 4 "Proxies")
        const char* e = std::getenv("DG_PROXY_REFRESH");  // developer knob
        int dev = 0, sms = 148;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        const int64_t autoint = std::min<int64_t>(128, std::max<int64_t>(8, D.n_part / ((int64_t)sms * 16)));
        P.px_refresh = e ? std::atoi(e) : (int)autoint;
    }
    if (accum && P.n_proxy) {
        // as many proxies as fit next to the rings in one CTA per SM (the top
        // ids are the highest-degree vertices, so a smaller H' is still the hubs)
        int dev = 0, sm_bytes = 0;
        cudaFuncAttributes fa{};
        CK(cudaGetDevice(&dev));
        CK(cudaDeviceGetAttribute(&sm_bytes, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev));
        CK(cudaFuncGetAttributes(&fa, fn));
        const int64_t room = sm_bytes - (int64_t)fa.sharedSizeBytes - (int64_t)gbuf_bytes<kAccWarps>();
        P.n_proxy = std::max<int64_t>(0, std::min<int64_t>(P.n_proxy, room / kPxBytes));
    }
    const size_t smem = accum ? gbuf_bytes<kAccWarps>() + (size_t)P.n_proxy * kPxBytes : 0;
    if (accum) P.e_coef = algo_k == DG_ADSORPTION ? W->e_coef : W->pr_coef;
    {
        const char* dl = std::getenv("DG_DELTA");  // bucket width knob; default: reading R-DELTA
        // clamped to INF: sat_add and the bucket advance assume operands <= INF
        const long long dv = dl ? std::atoll(dl) : (long long)S.delta;
        P.delta = (uint32_t)std::min<long long>(std::max<long long>(dv, 0), (long long)INF);
        const int64_t sd = sparse_div();
        if ((algo_k == DG_SSSP || algo_k == DG_BFS || algo_k == 100 || algo_k == 101 || algo_k == DG_PAGERANK ||
             algo_k == DG_ADSORPTION || algo_k == DG_WCC) && sd > 0 && D.M >= sparse_min_entries()) {
            int rc;
            const bool in = algo_k == 101;
            if ((rc = ensure_occ(W, D, S, in, err))) return rc;
            if (algo_k == DG_WCC) {  // both directions
                if ((rc = ensure_occ(W, D, S, true, err))) return rc;
                P.iocc_off = W->iocc_off;
                P.iocc = W->iocc;
            }
            P.occ_off = in ? W->iocc_off : W->occ_off;
            P.occ = in ? W->iocc : W->occ;
            P.occ_items = W->occ_items;
            const char* cwe = std::getenv("DG_SPARSE_CW");  // developer knob: 0 = separate e_idx / e_w loads
            if (algo_k == DG_SSSP && D.e_w && !(cwe && std::atoi(cwe) == 0)) {
                if (!W->cw_ok) {
                    int64_t bytes = 0;
                    if (!W->e_cw && (rc = dalloc(&W->e_cw, (size_t)D.M + kPad, bytes, err))) return rc;
                    cw_build_kernel<<<grid_1d(D.M + kPad), 256>>>(W->e_cw, D.e_idx, D.e_w, D.M + kPad);
                    CK(cudaGetLastError());
                    S.stats.kernel_launches++;
                    W->cw_ok = true;
                }
                P.e_cw = W->e_cw;
            }
            P.sparse_max = (uint32_t)std::min<int64_t>(D.n / 4, 0xFFFFFFFFll);
            P.sparse_occ = (uint32_t)std::min<int64_t>(D.M / sd, 0xFFFFFFFFll);
            const char* sw = std::getenv("DG_SPARSE_WALK");  // developer knob
            P.sparse_walk = sw ? std::max(1, std::atoi(sw)) : 4;
        }
        {
            const char* pf = std::getenv("DG_PROBE_FREE");  // developer knob: 0 = always probe, k > 1: out-edge share M/k
            int64_t pdiv = pf ? std::atoll(pf) : 4;
            if (pdiv == 1) pdiv = 4;  // 1: on, with the default share
            P.probe_free_occ = pdiv == 0 ? 0u : (uint32_t)std::min<int64_t>(std::max<int64_t>(D.M / std::max<int64_t>(pdiv, 1), 1), 0xFFFFFFFFll);
            P.probe_free_act = (uint32_t)std::min<int64_t>(D.n / 4, 0xFFFFFFFFll);
        }
        const char* hm = std::getenv("DG_HOT_MASTER_MB");  // developer knob (default 64 MB)
        P.hot_master_bytes = (uint64_t)(hm ? std::atof(hm) : 64.0) * (1ull << 20);
        const char* o = std::getenv("DG_PART_ORDER");
        P.part_order = o ? std::atoi(o) : 0;
        if (P.part_order > 1) {  // keep the map a permutation
            auto gcd = [](long long a, long long b) { while (b) { long long t2 = a % b; a = b; b = t2; } return a; };
            while (gcd(P.part_order, D.n_part) != 1) P.part_order++;
        }
    }
#ifdef DG_EXP
    if (const char* xe = std::getenv("DG_EXP")) P.exp = std::atoi(xe);
    if (P.exp & 96) {
        CK(cudaMalloc(&P.snap, sizeof(unsigned long long) * 2 * (D.n + 4)));
        CK(cudaMemset(P.snap, 0, sizeof(unsigned long long) * 2 * (D.n + 4)));
    }
#endif
    // developer trace (DG_TRACE): per-round timing and activity on stderr
    unsigned long long* trace = nullptr;
    constexpr int kTraceCap = 1 << 16;
    if (std::getenv("DG_TRACE") && cudaMalloc(&trace, sizeof(unsigned long long) * 4 * kTraceCap) == cudaSuccess) {
        cudaMemset(trace, 0, sizeof(unsigned long long) * 4 * kTraceCap);
        P.trace = trace;
        P.trace_cap = kTraceCap;
    }
    P.ctr_out = mr ? nullptr : W->ctr_host_dev;
    W->ctr_mirror_fresh = false;
    // min-plus walks of small graphs (< 2^21 path entries) run 2 CTAs per SM
    // instead of 3: the per-round grid barriers and dispatch are cheaper and
    // the fewer warps still cover the windows (R-MAT-16 SSSP)
    int per_sm = D.M < ((int64_t)1 << 21) ? 2 : 0;
    if (const char* ce = std::getenv("DG_MP_CTAS")) per_sm = std::atoi(ce);  // developer knob: min-plus CTAs per SM
    int rc = coop_launch(W, fn, P, S, err, smem, accum ? kAccWarps * 32 : kBlock, accum ? 0 : per_sm);
    if (!rc && P.ctr_out) W->ctr_mirror_fresh = true;
    if (P.snap) cudaFree(P.snap);
    if (trace) {
        std::vector<unsigned long long> h(4 * (size_t)kTraceCap);
        cudaMemcpy(h.data(), trace, sizeof(unsigned long long) * h.size(), cudaMemcpyDeviceToHost);
        cudaFree(trace);
        for (int r = 0; r < kTraceCap && h[4 * r]; r++) {
            const unsigned long long prev = r ? h[4 * (r - 1)] : 0ull;  // round 0: no reference
            fprintf(stderr, "[trace] algo %d round %d: %.1f us, signalled-in %llu, %s, out-edges %llu\n", algo_k, r,
                    prev ? (h[4 * r] - prev) / 1e3 : 0.0, h[4 * r + 1], h[4 * r + 2] ? "dense" : "sparse",
                    h[4 * r + 3]);
        }
    }
    return rc;
}

int launch_vertex(DevWork* W, const DevLayout& D, int algo, int rounds, RunState& S, std::string& err) {
    KParams P = make_params(D, W);
    P.eps = (float)S.eps;
    P.max_rounds = rounds;
    void* fn = algo == DG_PAGERANK ? (void*)vertex_kernel<DG_PAGERANK>
             : algo == DG_BFS ? (void*)vertex_kernel<DG_BFS>
             : algo == DG_WCC ? (void*)vertex_kernel<DG_WCC> : (void*)vertex_kernel<DG_SSSP>;
    if (algo == DG_WCC) {  // labels cross every edge in both directions
        P.row_ptr = D.srow_ptr;
        P.col = D.scol;
    }
    return coop_launch(W, fn, P, S, err);
}

int init_states(DevWork* W, const DevLayout& D, RunState& S, std::string& err) {
    const int algo = S.algo;
    const int g = grid_1d(D.n);
    Counters c{};
    if (S.mode == DG_MODE_VERTEX) {
        // frontier: the source (SSSP/BFS) or every vertex (PageRank)
        if (algo == DG_PAGERANK) {
            init_pr_kernel<<<g, 256>>>(W->vs_f, D.outdeg, D.n, (float)S.param);
            fill_iota_kernel<<<g, 256>>>(W->vlist[0], D.n);
            c.active[0] = (unsigned)D.n;
            S.stats.kernel_launches += 2;
        } else if (algo == DG_WCC) {  // every vertex starts with its own label, all in the frontier
            init_u_kernel<<<g, 256>>>(W->vs_u, W->vstamp, D.orig, D.n, algo, 0);
            fill_iota_kernel<<<g, 256>>>(W->vlist[0], D.n);
            c.active[0] = (unsigned)D.n;
            S.stats.kernel_launches += 2;
        } else {
            init_u_kernel<<<g, 256>>>(W->vs_u, W->vstamp, D.orig, D.n, algo, S.source);
            int32_t s = (int32_t)S.source;
            CK(cudaMemcpy(W->vlist[0], &s, sizeof(int32_t), cudaMemcpyHostToDevice));
            c.active[0] = 1;
            S.stats.kernel_launches += 1;
        }
        CK(cudaGetLastError());
        return write_counters(W, c, err, &S);
    }
    c.minval[0] = c.minval[1] = INF;
    if (algo == DG_SSSP || algo == DG_BFS) {
        // one launch: distances, both bitmaps (the source signalled) and the counters
        c.minval[0] = 0;  // round 0's bucket starts at the source's distance
        c.active[0] = 1;
        init_minplus_kernel<<<grid_1d(std::max<int64_t>(D.n, 2 * W->nw)), 256>>>(W->vs_u, W->vstamp, D.n, S.source,
                                                                                W->bits, 2 * W->nw, W->ctr, c);
        S.stats.kernel_launches += 1;
        CK(cudaGetLastError());
        return DG_OK;
    }
    CK(cudaMemsetAsync(W->bits, 0, sizeof(uint32_t) * 2 * W->nw));
    {
        if (algo == DG_WCC) {
            init_u_kernel<<<g, 256>>>(W->vs_u, W->vstamp, D.orig, D.n, algo, 0);
        } else {
            init_acc_kernel<<<g, 256>>>(W->vs_t, W->sigma, algo == DG_ADSORPTION ? W->ads_base : nullptr, D.n,
                                        (float)S.param);
            if (algo == DG_PAGERANK && W->pr_coef_d != S.param) {  // per-entry d/outdeg, cached per damping
                int64_t bytes = 0;
                int rc;
                if (!W->pr_coef && (rc = dalloc(&W->pr_coef, D.M + kPad, bytes, err))) return rc;
                CK(cudaMemsetAsync(W->pr_coef, 0, sizeof(float) * (D.M + kPad)));
                pr_coef_kernel<<<grid_1d(D.M), 256>>>(W->pr_coef, D.e_idx, D.outdeg, (float)S.param, D.M);
                W->pr_coef_d = S.param;
                S.stats.kernel_launches++;
            }
            CK(cudaMemsetAsync(W->s_val, 0, sizeof(unsigned long long) * (D.M + kPad)));
        }
        bits_all_kernel<<<grid_1d(W->nw), 256>>>(W->bits, W->nw, D.n);
        c.active[0] = (unsigned)D.n;
        S.stats.kernel_launches += 2;
    }
    CK(cudaGetLastError());
    return write_counters(W, c, err, &S);
}

int collect_stats(DevWork* W, RunState& S, std::string& err, Counters* out = nullptr, bool mirror = false) {
    Counters c;
    int rc;
    if (mirror && W->ctr_mirror_fresh && W->ctr_host) {  // written by the path kernel that just completed
        std::memcpy(&c, (const void*)W->ctr_host, sizeof(Counters));
        W->ctr_mirror_fresh = false;
    } else if ((rc = read_counters(W, c, err))) {
        return rc;
    }
    if (out) *out = c;
    S.stats.rounds += c.round - (int)S.round;
    S.round = c.round;
    S.stats.vertex_updates = (int64_t)c.updates;
    S.stats.edges_processed = (int64_t)c.edges;
    S.stats.units_processed = (int64_t)c.units;
    S.stats.entries_processed = (int64_t)c.entries;
    S.stats.csr_edges = (int64_t)c.pushes;
    S.stats.dense_rounds = (int64_t)c.dense_rounds;
    return DG_OK;
}

// SCC by colouring: repeat { forward min-colour rounds over
// unassigned vertices; roots = vertices keeping their own id; backward
// reachability inside each colour from its root; reached vertices form the
// SCC labelled by the colour (= smallest id in the SCC) }.
int run_scc(DevWork* W, const DevLayout& D, RunState& S, int64_t max_rounds, std::string& err) {
    int rc;
    int64_t bytes = 0;
    if (!W->scc_label) {
        if ((rc = dalloc(&W->scc_label, D.n + 1, bytes, err))) return rc;
        if ((rc = dalloc(&W->scc_mark, D.n + 1, bytes, err))) return rc;
        if ((rc = dalloc(&W->remaining, 1, bytes, err))) return rc;
    }
    const int g = grid_1d(D.n);
    CK(cudaMemset(W->scc_label, 0xff, sizeof(int32_t) * D.n));
    Counters tot{};
    int64_t total_rounds = 0;
    const int rounds = (int)std::min<int64_t>(max_rounds, 1 << 30);
    const bool verbose = std::getenv("DG_VERBOSE") != nullptr;
    int32_t rem = (int32_t)D.n;
    for (int64_t it = 0;; it++) {
        // forward colouring: every unassigned vertex starts with its own id, all signalled
        scc_init_kernel<<<g, 256>>>(W->vs_u, W->scc_label, D.orig, W->scc_mark, D.n);
        CK(cudaMemsetAsync(W->bits, 0, sizeof(uint32_t) * 2 * W->nw));
        scc_bits_kernel<<<grid_1d(W->nw), 256>>>(W->scc_label, D.n, W->bits, W->nw);
        Counters c0{};
        c0.active[0] = (unsigned)rem;
        if ((rc = write_counters(W, c0, err, &S))) return rc;
        S.stats.kernel_launches += 2;
        if ((rc = launch_path(W, D, 100, rounds, S, err))) return rc;
        Counters c1;
        if ((rc = read_counters(W, c1, err))) return rc;
        if (c1.active[c1.round & 1] != 0) {  // colours not final: roots would be wrong
            err = "SCC forward colouring: max_rounds reached before convergence";
            return DG_ENOCONV;
        }
        // backward reachability from the roots within their colours
        CK(cudaMemsetAsync(W->bits, 0, sizeof(uint32_t) * 2 * W->nw));
        Counters c2{};
        if ((rc = write_counters(W, c2, err, &S))) return rc;
        scc_roots_kernel<<<g, 256>>>(W->vs_u, W->scc_label, D.orig, W->scc_mark, D.n, W->bits, W->ctr);
        S.stats.kernel_launches += 1;
        if ((rc = launch_path(W, D, 101, rounds, S, err))) return rc;
        Counters c3;
        if ((rc = read_counters(W, c3, err))) return rc;
        if (c3.active[c3.round & 1] != 0) {
            err = "SCC backward reachability: max_rounds reached before convergence";
            return DG_ENOCONV;
        }
        total_rounds += c1.round + c3.round;
        tot.updates += c1.updates + c3.updates;
        tot.edges += c1.edges + c3.edges;
        tot.units += c1.units + c3.units;
        tot.entries += c1.entries + c3.entries;
        tot.dense_rounds += c1.dense_rounds + c3.dense_rounds;
        CK(cudaMemset(W->remaining, 0, sizeof(int32_t)));
        scc_assign_kernel<<<g, 256>>>(W->vs_u, W->scc_label, W->scc_mark, D.n, W->remaining);
        S.stats.kernel_launches += 1;
        CK(cudaMemcpy(&rem, W->remaining, sizeof(int32_t), cudaMemcpyDeviceToHost));
        S.stats.outer_iterations = it + 1;
        if (verbose)
            fprintf(stderr, "[dg] scc iteration %lld: forward %d rounds, backward %d rounds, %d unassigned\n",
                    (long long)it, c1.round, c3.round, rem);
        if (rem == 0) break;
        if (it > D.n) { err = "SCC colouring did not terminate"; return DG_ENOCONV; }
    }
    S.stats.rounds = total_rounds;
    S.stats.vertex_updates = (int64_t)tot.updates;
    S.stats.edges_processed = (int64_t)tot.edges;
    S.stats.units_processed = (int64_t)tot.units;
    S.stats.entries_processed = (int64_t)tot.entries;
    S.stats.dense_rounds = (int64_t)tot.dense_rounds;
    return DG_OK;
}

}  // namespace

// ------------------------------------------------------------------ API glue
int dev_select(int device, std::string& err) {
    int cnt = 0;
    if (cudaGetDeviceCount(&cnt) != cudaSuccess || cnt == 0) {
        err = "no CUDA device available (the DiGraph hot path has no CPU fallback)";
        return DG_ENOCUDA;
    }
    if (device < 0 || device >= cnt) { err = "device ordinal out of range"; return DG_EINVAL; }
    CK(cudaSetDevice(device));
    return DG_OK;
}

// dg_upload: the per-vertex arrays every run needs (out-degrees and both id
// maps, internal ids); the CSR (vertex-centric ablation, Adsorption weights)
// and the path-edge weights (SSSP) follow on first use (dev_ensure_parts), so
// a run moves only the bytes its algorithm reads.
int dev_upload_csr(DevLayout& D, const HostCSR& g, const HostLayout& L, std::string& err) {
    int dev_count = 0;
    if (cudaGetDeviceCount(&dev_count) != cudaSuccess || dev_count == 0) {
        err = "no CUDA device available (the DiGraph hot path has no CPU fallback)";
        return DG_ENOCUDA;
    }
    int rc;
    D.n = g.n; D.m = g.m;
    D.h2d_bytes = 0;
    D.csr_ok = D.ew_ok = false;
    g_h2d_counter = &D.h2d_bytes;
    g_pin_list = &D.pinned;
    if ((rc = dalloc_once(&D.outdeg, g.n + 1, D.bytes, err))) return rc;
    if ((rc = dalloc_once(&D.new_id, g.n + 1, D.bytes, err))) return rc;
    if ((rc = dalloc_once(&D.orig, g.n + 1, D.bytes, err))) return rc;
    if ((rc = h2d(D.outdeg, L.poutdeg.data(), g.n, err))) return rc;
    if ((rc = h2d(D.new_id, L.new_id.data(), g.n, err))) return rc;
    if ((rc = h2d(D.orig, L.orig.data(), g.n, err))) return rc;
    D.n_proxy = L.n_proxy;
    return DG_OK;
}

int dev_ensure_parts(DevLayout& D, const HostCSR& g, const HostLayout& L, bool need_csr, bool need_ew, bool need_sym,
                     std::string& err) {
    int rc;
    g_h2d_counter = &D.h2d_bytes;
    g_pin_list = &D.pinned;
    if (need_csr && !D.csr_ok) {  // the CSR in internal ids (HostLayout)
        if ((rc = dalloc_once(&D.row_ptr, g.n + 1, D.bytes, err))) return rc;
        if ((rc = dalloc_once(&D.col, g.m + kPad, D.bytes, err))) return rc;
        if ((rc = h2d(D.row_ptr, L.prow_ptr.data(), g.n + 1, err))) return rc;
        if ((rc = h2d(D.col, L.pcol.data(), g.m, err))) return rc;
        if (g.has_w) {
            if ((rc = dalloc_once(&D.w, g.m + kPad, D.bytes, err))) return rc;
            if ((rc = h2d(D.w, L.pw.data(), g.m, err))) return rc;
        }
        D.csr_ok = true;
    }
    if (need_sym && !D.sym_ok) {  // the CSR of both directions (dg_api.cpp builds it on the host)
        const int64_t ms = (int64_t)L.scol.size();
        if ((rc = dalloc_once(&D.srow_ptr, g.n + 1, D.bytes, err))) return rc;
        if ((rc = dalloc_once(&D.scol, ms + kPad, D.bytes, err))) return rc;
        if ((rc = h2d(D.srow_ptr, L.srow_ptr.data(), g.n + 1, err))) return rc;
        if ((rc = h2d(D.scol, L.scol.data(), ms, err))) return rc;
        D.sym_ok = true;
    }
    if (need_ew && !D.ew_ok) {
        if ((rc = dalloc_once(&D.e_w, D.M + kPad, D.bytes, err))) return rc;
        CK(cudaMemset(D.e_w + D.M, 0, sizeof(int32_t) * kPad));
        if ((rc = h2d(D.e_w, L.e_w.data(), D.M, err))) return rc;
        D.ew_ok = true;
    }
    g_h2d_counter = nullptr;
    g_pin_list = nullptr;
    return DG_OK;
}

int dev_upload_layout(DevLayout& D, const HostLayout& L, std::string& err) {
    int rc;
    g_h2d_counter = &D.h2d_bytes;
    g_pin_list = &D.pinned;
    D.M = (int64_t)L.e_idx.size();
    if (D.M + kPad + 256 >= (int64_t)0xFFFFFFFFll) {  // the kernels use 32-bit entry offsets
        err = "layout has >= 2^32 path entries on one rank; use more ranks";
        return DG_EINVAL;
    }
    D.n_part = (int64_t)L.part_off.size() - 1;
    D.max_part = 0;
    for (int64_t q = 0; q < D.n_part; q++) D.max_part = std::max(D.max_part, L.part_off[q + 1] - L.part_off[q]);
    D.n_bnd = (int64_t)L.boundary.size();
    if ((rc = dalloc_once(&D.e_idx, D.M + kPad, D.bytes, err))) return rc;
    if ((rc = dalloc_once(&D.part_off, D.n_part + 1, D.bytes, err))) return rc;
    if ((rc = dalloc_once(&D.bnd, D.n_bnd + 1, D.bytes, err))) return rc;
    if ((rc = dalloc_once(&D.bnd_hold, D.n_bnd + 1, D.bytes, err))) return rc;
    CK(cudaMemset(D.e_idx + D.M, 0, sizeof(uint32_t) * kPad));
    if ((rc = h2d(D.e_idx, L.e_idx.data(), D.M, err))) return rc;
    if ((rc = h2d(D.part_off, L.part_off.data(), D.n_part + 1, err))) return rc;
    if ((rc = h2d(D.bnd, L.boundary.data(), D.n_bnd, err))) return rc;
    if ((rc = h2d(D.bnd_hold, (const unsigned long long*)L.bnd_hold.data(), D.n_bnd, err))) return rc;
    CK(cudaDeviceSynchronize());
    g_h2d_counter = nullptr;
    g_pin_list = nullptr;
    return DG_OK;
}

void dev_unpin_all(DevLayout& D) {
    for (void* q : D.pinned) cudaHostUnregister(q);
    D.pinned.clear();
    cudaGetLastError();
}

void dev_free_layout(DevLayout& D, bool csr_too) {
    dfree(D.e_idx); dfree(D.e_w); dfree(D.part_off); dfree(D.bnd); dfree(D.bnd_hold);
    if (csr_too) {
        dfree(D.row_ptr); dfree(D.col); dfree(D.w); dfree(D.outdeg); dfree(D.new_id); dfree(D.orig);
        dfree(D.srow_ptr); dfree(D.scol);
        D.sym_ok = false;
    }
    D.bytes = 0;
    D.M = D.n_part = D.n_bnd = 0;
    D.csr_ok = D.ew_ok = false;
}

void dev_free_work(DevWork*& W) {
    if (!W) return;
    dfree(W->vs_u); dfree(W->vstamp); dfree(W->vs_f); dfree(W->vs_t); dfree(W->sigma); dfree(W->s_val); dfree(W->bnd_base);
    dfree(W->e_coef); dfree(W->pr_coef); dfree(W->ads_base); dfree(W->bits); dfree(W->vlist[0]); dfree(W->vlist[1]);
    if (W->ctr_host) cudaFreeHost(W->ctr_host);
    W->ctr_host = W->ctr_host_dev = nullptr;
    if (W->host_stage) cudaFreeHost(W->host_stage);
    W->host_stage = nullptr;
    W->host_stage_n = 0;
    dfree(W->ctr); dfree(W->dsum); dfree(W->qtick); dfree(W->scc_label); dfree(W->scc_mark); dfree(W->remaining); dfree(W->out_stage);
    dfree(W->occ_off); dfree(W->occ); dfree(W->occ_items); dfree(W->e_cw); dfree(W->iocc_off); dfree(W->iocc); dfree(W->occ_cur);
    if (W->cub_tmp) cudaFree(W->cub_tmp);
    if (W->ev0) cudaEventDestroy(W->ev0);
    if (W->ev1) cudaEventDestroy(W->ev1);
    if (W->kev0) cudaEventDestroy(W->kev0);
    if (W->kev1) cudaEventDestroy(W->kev1);
    delete W;
    W = nullptr;
}

void dev_layout_changed(DevWork* W) {
    if (!W) return;
    W->pr_coef_d = -1.0;
    W->occ_ok = W->iocc_ok = false;  // rebuilt on next use (allocations kept: same n, M)
    W->cw_ok = false;
}

int dev_set_vertex_params(DevWork*& W, const DevLayout& D, const double* p_inj, const double* p_cont,
                          const double* inj, const float* wsum_h, std::string& err) {
    int rc;
    if ((rc = ensure_work(W, D, err))) return rc;
    if (!D.e_w) { err = "Adsorption needs the path-edge weights on the device"; return DG_EINVAL; }
    int64_t bytes = 0;
    if (!W->ads_base) {
        if ((rc = dalloc(&W->ads_base, D.n + 1, bytes, err))) return rc;
        if ((rc = dalloc(&W->e_coef, D.M + kPad, bytes, err))) return rc;
    }
    std::vector<float> base(D.n), pc(D.n);
    for (int64_t v = 0; v < D.n; v++) { base[v] = (float)(p_inj[v] * inj[v]); pc[v] = (float)p_cont[v]; }
    float *pcont = nullptr, *wsum = nullptr;
    if ((rc = dalloc(&pcont, D.n + 1, bytes, err))) return rc;
    if ((rc = dalloc(&wsum, D.n + 1, bytes, err))) { cudaFree(pcont); return rc; }
    rc = h2d(W->ads_base, base.data(), D.n, err);
    if (!rc) rc = h2d(pcont, pc.data(), D.n, err);
    if (!rc) rc = h2d(wsum, wsum_h, D.n, err);  // W(u), summed on the host at preprocessing
    if (!rc) {
        cudaMemset(W->e_coef, 0, sizeof(float) * (D.M + kPad));
        ads_coef_kernel<<<grid_1d(D.M), 256>>>(W->e_coef, D.e_idx, D.e_w, pcont, wsum, D.M);
        cudaError_t e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { err = cudaGetErrorString(e); rc = DG_ENOCUDA; }
    }
    cudaFree(pcont);
    cudaFree(wsum);
    if (!rc) W->have_params = true;
    return rc;
}

int dev_run(DevWork*& W, const DevLayout& D, RunState& S, int64_t max_rounds, std::string& err) {
    int rc;
    if ((rc = ensure_work(W, D, err))) return rc;
    if (S.algo == DG_ADSORPTION && !W->have_params) {
        err = "Adsorption needs dg_set_vertex_params first";
        return DG_EINVAL;
    }
    CK(cudaEventRecord(W->ev0));
    if (S.algo == DG_SCC) {
        if ((rc = run_scc(W, D, S, max_rounds, err))) return rc;
    } else {
        if ((rc = init_states(W, D, S, err))) return rc;
        const int rounds = (int)std::min<int64_t>(max_rounds, 1 << 30);
        W->defer_kernel_time = true;
        W->kernel_time_pending = false;
        rc = S.mode == DG_MODE_VERTEX ? launch_vertex(W, D, S.algo, rounds, S, err)
                                      : launch_path(W, D, S.algo, rounds, S, err);
        W->defer_kernel_time = false;
        if (rc) return rc;
    }
    CK(cudaEventRecord(W->ev1));
    CK(cudaEventSynchronize(W->ev1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, W->ev0, W->ev1));
    S.stats.time_ms = ms;
    if (W->kernel_time_pending) {  // kev1 precedes ev1 in the stream: complete
        float kms = 0;
        CK(cudaEventElapsedTime(&kms, W->kev0, W->kev1));
        S.stats.kernel_ms += kms;
        W->kernel_time_pending = false;
    }
    if (S.algo != DG_SCC) {
        Counters c;
        // the mirror is valid only right after a single-rank path launch of this run
        if ((rc = collect_stats(W, S, err, &c, S.mode != DG_MODE_VERTEX))) return rc;
        if (c.active[c.round & 1] != 0) {
            err = "max_rounds reached before convergence";
            return DG_ENOCONV;
        }
    }
    return DG_OK;
}

// ---- multi-rank SCC (dg_run_begin(DG_SCC) / dg_scc_phase / dg_scc_assign):
// the colouring iterations of run_scc with every phase a multi-rank run --
// forward colouring exchanges colours with MIN, backward reachability
// exchanges marks (MIN of 0 = marked / 1 = not, i.e. OR).  A vertex on none
// of this rank's paths is assigned its own original id at the start: the
// owning ranks' labels are <= it, so a MIN over ranks gives every vertex its
// SCC label, and a vertex on no rank's paths (no edges) is its own SCC.
namespace {
__global__ void scc_present_kernel(const uint32_t* e_idx, int64_t M, uint8_t* mark) {
    GRID_STRIDE(i, M) mark[e_idx[i] & kVMask] = 1;
}
__global__ void scc_label_init_kernel(int32_t* label, uint8_t* mark, const int32_t* orig, int64_t n) {
    GRID_STRIDE(v, n) {
        label[v] = mark[v] ? -1 : orig[v];
        mark[v] = 0;
    }
}
__global__ void scc_count_kernel(const int32_t* label, int64_t n, int32_t* remaining) {
    int cnt = 0;
    GRID_STRIDE(v, n) cnt += label[v] < 0;
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(remaining, cnt);
}
// the device counters of the phase that just ran, added to the run's statistics
int fold_counters(DevWork* W, RunState& S, std::string& err) {
    Counters c;
    int rc;
    if ((rc = read_counters(W, c, err))) return rc;
    S.stats.rounds += c.round;
    S.stats.vertex_updates += (int64_t)c.updates;
    S.stats.edges_processed += (int64_t)c.edges;
    S.stats.units_processed += (int64_t)c.units;
    S.stats.entries_processed += (int64_t)c.entries;
    S.stats.dense_rounds += (int64_t)c.dense_rounds;
    return write_counters(W, Counters{}, err);
}
}  // namespace

// the kernel algorithm of a run (SCC phases: 100 forward colouring, 101 backward marks)
int launch_algo(const RunState& S) { return S.algo == DG_SCC ? (S.scc_phase == 1 ? 101 : 100) : S.algo; }
// the replicated mark array of an SCC backward phase (else null: MIN over vs_u)
uint8_t* scc_marks(DevWork* W, const RunState& S) { return S.algo == DG_SCC && S.scc_phase == 1 ? W->scc_mark : nullptr; }

int dev_scc_begin(DevWork*& W, const DevLayout& D, RunState& S, std::string& err) {
    int rc;
    if ((rc = ensure_work(W, D, err))) return rc;
    int64_t bytes = 0;
    if (!W->scc_label) {
        if ((rc = dalloc(&W->scc_label, D.n + 1, bytes, err))) return rc;
        if ((rc = dalloc(&W->scc_mark, D.n + 1, bytes, err))) return rc;
        if ((rc = dalloc(&W->remaining, 1, bytes, err))) return rc;
    }
    CK(cudaMemset(W->scc_mark, 0, D.n + 1));
    if (D.M) scc_present_kernel<<<grid_1d(D.M), 256>>>(D.e_idx, D.M, W->scc_mark);
    scc_label_init_kernel<<<grid_1d(D.n), 256>>>(W->scc_label, W->scc_mark, D.orig, D.n);
    CK(cudaGetLastError());
    S.scc_phase = -1;
    S.stats.kernel_launches += 2;
    if ((rc = write_counters(W, Counters{}, err))) return rc;
    CK(cudaEventRecord(W->ev0));
    return DG_OK;
}

int dev_scc_phase(DevWork* W, const DevLayout& D, RunState& S, int phase, int64_t* active, std::string& err) {
    if (!W || !W->scc_label) { err = "dg_scc_phase: no SCC run in progress"; return DG_EINVAL; }
    int rc;
    if ((rc = fold_counters(W, S, err))) return rc;
    CK(cudaMemsetAsync(W->bits, 0, sizeof(uint32_t) * 2 * W->nw));
    const int g = grid_1d(D.n);
    Counters c{};
    if (phase == 0) {  // forward colouring: unassigned vertices start with their own id, all signalled
        scc_init_kernel<<<g, 256>>>(W->vs_u, W->scc_label, D.orig, W->scc_mark, D.n);
        scc_bits_kernel<<<grid_1d(W->nw), 256>>>(W->scc_label, D.n, W->bits, W->nw);
        CK(cudaMemset(W->remaining, 0, sizeof(int32_t)));
        scc_count_kernel<<<g, 256>>>(W->scc_label, D.n, W->remaining);
        int32_t rem = 0;
        CK(cudaMemcpy(&rem, W->remaining, sizeof(int32_t), cudaMemcpyDeviceToHost));
        c.active[0] = (unsigned)rem;
        if ((rc = write_counters(W, c, err))) return rc;
        *active = rem;
        S.stats.kernel_launches += 3;
    } else {  // backward reachability from the roots (vertices keeping their own id)
        scc_roots_kernel<<<g, 256>>>(W->vs_u, W->scc_label, D.orig, W->scc_mark, D.n, W->bits, W->ctr);
        S.stats.kernel_launches += 1;
        if ((rc = read_counters(W, c, err))) return rc;
        *active = c.active[0];
    }
    CK(cudaGetLastError());
    S.scc_phase = phase;
    S.round = 0;
    return DG_OK;
}

int dev_scc_assign(DevWork* W, const DevLayout& D, RunState& S, int64_t* remaining, std::string& err) {
    if (!W || !W->scc_label || S.scc_phase != 1) { err = "dg_scc_assign: after a backward phase only"; return DG_EINVAL; }
    int rc;
    if ((rc = fold_counters(W, S, err))) return rc;
    CK(cudaMemset(W->remaining, 0, sizeof(int32_t)));
    scc_assign_kernel<<<grid_1d(D.n), 256>>>(W->vs_u, W->scc_label, W->scc_mark, D.n, W->remaining);
    int32_t rem = 0;
    CK(cudaMemcpy(&rem, W->remaining, sizeof(int32_t), cudaMemcpyDeviceToHost));
    *remaining = rem;
    S.stats.kernel_launches += 1;
    S.stats.outer_iterations++;
    S.scc_phase = -1;
    return DG_OK;
}

int dev_run_begin(DevWork*& W, const DevLayout& D, RunState& S, std::string& err) {
    if (S.algo == DG_SCC) return dev_scc_begin(W, D, S, err);
    int rc;
    if ((rc = ensure_work(W, D, err))) return rc;
    if (S.algo == DG_ADSORPTION && !W->have_params) { err = "Adsorption needs dg_set_vertex_params first"; return DG_EINVAL; }
    if ((rc = init_states(W, D, S, err))) return rc;
    if ((S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION) && D.n_bnd)
        init_base_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_t, D.bnd, D.n_bnd, W->bnd_base);
    CK(cudaGetLastError());
    CK(cudaEventRecord(W->ev0));
    return DG_OK;
}

int dev_rounds(DevWork* W, const DevLayout& D, RunState& S, int64_t max_rounds, int64_t* active, std::string& err) {
    int rc;
    if (S.algo == DG_SCC && S.scc_phase < 0) { err = "dg_rounds: SCC run without a phase (dg_scc_phase)"; return DG_EINVAL; }
    if ((rc = launch_path(W, D, launch_algo(S), (int)std::min<int64_t>(max_rounds, 1 << 30), S, err))) return rc;
    Counters c;
    if ((rc = read_counters(W, c, err))) return rc;
    *active = c.active[c.round & 1];
    return DG_OK;
}

int dev_boundary_pack(DevWork* W, const DevLayout& D, RunState& S, void* buf, std::string& err) {
    if (!D.n_bnd) return DG_OK;
    if (S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION)
        pack_sum_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_t, D.bnd, D.n_bnd, W->bnd_base, (unsigned long long*)buf);
    else
        pack_min_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_u, scc_marks(W, S), D.bnd, D.n_bnd, (uint32_t*)buf);
    S.stats.kernel_launches++;
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    return DG_OK;
}

int dev_boundary_unpack(DevWork* W, const DevLayout& D, RunState& S, const void* buf, int64_t* active,
                        std::string& err) {
    Counters c;
    int rc;
    if ((rc = read_counters(W, c, err))) return rc;
    const int slot = c.round & 1;  // the bitmap the next local round reads
    if (D.n_bnd) {
        uint32_t* b = W->bits + (int64_t)slot * W->nw;
        if (S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION)
            unpack_sum_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_t, W->sigma, D.bnd, D.n_bnd, W->bnd_base,
                                                         (const unsigned long long*)buf,
                                                         (unsigned long long)(S.eps * 4294967296.0), b, W->ctr,
                                                         slot);
        else
            unpack_min_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_u, scc_marks(W, S), W->scc_label, D.bnd, D.n_bnd,
                                                         (const uint32_t*)buf, b, W->ctr, slot);
        S.stats.kernel_launches++;
        CK(cudaGetLastError());
    }
    if ((rc = read_counters(W, c, err))) return rc;
    *active = c.active[slot];
    return DG_OK;
}

struct P2P {
    int world = 0, rank = 0;
    int64_t nb = 0;
    unsigned long long epoch = 0;   // exchanges done (identical on every rank)
    unsigned char* own = nullptr;   // this rank's exchange region (cudaMalloc)
    unsigned char* peer[kP2PMaxRanks] = {};  // every rank's region in this address space (own included)
    uint32_t* last = nullptr;       // fused runs, MIN: reduced boundary values of the last exchange
    bool opened = false;
};

int dev_p2p_alloc(P2P*& X, const DevLayout& D, int world, int rank, void* handle, std::string& err) {
    if (world < 2 || world > kP2PMaxRanks || rank < 0 || rank >= world) {
        err = "p2p: world must be 2.." + std::to_string(kP2PMaxRanks) + " and 0 <= rank < world";
        return DG_EINVAL;
    }
    dev_p2p_free(X);
    X = new P2P();
    X->world = world;
    X->rank = rank;
    X->nb = D.n_bnd;
    const size_t bytes = kP2PHeader + 2 * sizeof(unsigned long long) * (size_t)std::max<int64_t>(D.n_bnd, 1);
    CK(cudaMalloc(&X->own, bytes));
    CK(cudaMemset(X->own, 0, bytes));  // epochs 0 before any peer can see the region
    CK(cudaDeviceSynchronize());
    cudaIpcMemHandle_t h;
    CK(cudaIpcGetMemHandle(&h, X->own));
    std::memcpy(handle, &h, sizeof(h));
    return DG_OK;
}

int dev_p2p_open(P2P* X, const void* handles, std::string& err) {
    if (!X) { err = "p2p: dg_p2p_alloc first"; return DG_EINVAL; }
    for (int r = 0; r < X->world; r++) {
        if (r == X->rank) { X->peer[r] = X->own; continue; }
        if (X->peer[r]) continue;
        cudaIpcMemHandle_t h;
        std::memcpy(&h, (const unsigned char*)handles + (size_t)r * sizeof(h), sizeof(h));
        void* ptr = nullptr;
        CK(cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess));
        X->peer[r] = (unsigned char*)ptr;
    }
    X->opened = true;
    return DG_OK;
}

void dev_p2p_free(P2P*& X) {
    if (!X) return;
    for (int r = 0; r < X->world; r++)
        if (X->peer[r] && r != X->rank) cudaIpcCloseMemHandle(X->peer[r]);
    if (X->own) cudaFree(X->own);
    if (X->last) cudaFree(X->last);
    delete X;
    X = nullptr;
}

int dev_boundary_exchange(DevWork* W, const DevLayout& D, RunState& S, P2P* X, int64_t* active, std::string& err) {
    if (!X || !X->opened) { err = "dg_boundary_exchange: peers not opened (dg_p2p_open)"; return DG_EINVAL; }
    if (X->nb != D.n_bnd) { err = "dg_boundary_exchange: layout changed since dg_p2p_alloc"; return DG_EINVAL; }
    Counters c;
    int rc;
    if ((rc = read_counters(W, c, err))) return rc;
    const int slot = c.round & 1;  // the bitmap the next local round reads
    const unsigned long long e = ++X->epoch;
    const size_t off = kP2PHeader + (size_t)(e & 1) * sizeof(unsigned long long) * (size_t)std::max<int64_t>(D.n_bnd, 1);
    PeerSlots flags{}, slots{};
    for (int r = 0; r < X->world; r++) {
        flags.p[r] = X->peer[r];
        slots.p[r] = X->peer[r] + off;
    }
    const bool sum = S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION;
    unsigned long long* mine = (unsigned long long*)(X->own + off);
    if (D.n_bnd) {
        if (sum)
            p2p_pack_sum_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_t, D.bnd, D.bnd_hold, X->rank, D.n_bnd, W->bnd_base, mine);
        else
            p2p_pack_min_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_u, scc_marks(W, S), D.bnd, D.bnd_hold, X->rank, D.n_bnd,
                                                           mine);
    }
    unsigned long long* own_flags = (unsigned long long*)X->own;
    p2p_signal_wait_kernel<<<1, 32>>>(flags, X->world, X->rank, e, own_flags, 60ull * 1000000000ull);
    if (D.n_bnd) {
        uint32_t* b = W->bits + (int64_t)slot * W->nw;
        if (sum)
            p2p_reduce_sum_kernel<<<grid_1d(D.n_bnd), 256>>>(slots, X->rank, W->vs_t, W->sigma, D.bnd, D.bnd_hold,
                                                             D.n_bnd, W->bnd_base,
                                                             (unsigned long long)(S.eps * 4294967296.0), b, W->ctr, slot);
        else
            p2p_reduce_min_kernel<<<grid_1d(D.n_bnd), 256>>>(slots, X->rank, W->vs_u, scc_marks(W, S), W->scc_label,
                                                             D.bnd, D.bnd_hold, D.n_bnd, b, W->ctr, slot);
    }
    S.stats.kernel_launches += D.n_bnd ? 3 : 1;
    CK(cudaGetLastError());
    unsigned long long timed_out = 0;
    CK(cudaMemcpy(&timed_out, own_flags + kP2PErr, sizeof(timed_out), cudaMemcpyDeviceToHost));
    if (timed_out) { err = "dg_boundary_exchange: a peer did not arrive within 60 s"; return DG_ETIMEOUT; }
    if ((rc = read_counters(W, c, err))) return rc;
    *active = c.active[slot];
    return DG_OK;
}

// A whole multi-rank run in one launch per rank: the exchanges (every
// `local_rounds` rounds, or as soon as this rank has no work) and the global
// termination test run inside path_kernel (mr_exchange).
int dev_run_fused(DevWork* W, const DevLayout& D, RunState& S, P2P* X, int64_t local_rounds, int64_t max_rounds,
                  int64_t* exchanges, int64_t* converged, std::string& err) {
    if (!X || !X->opened) { err = "dg_run_fused: peers not opened (dg_p2p_open)"; return DG_EINVAL; }
    if (X->nb != D.n_bnd) { err = "dg_run_fused: layout changed since dg_p2p_alloc"; return DG_EINVAL; }
    if (S.algo == DG_SCC && S.scc_phase < 0) { err = "dg_run_fused: SCC run without a phase (dg_scc_phase)"; return DG_EINVAL; }
    const size_t nbs = (size_t)std::max<int64_t>(D.n_bnd, 1);
    if (!X->last) CK(cudaMalloc(&X->last, sizeof(uint32_t) * nbs));
    CK(cudaMemset(X->last, 0xFF, sizeof(uint32_t) * nbs));  // differs from every state: the first exchange is dirty
    MultiRank M{};
    for (int r = 0; r < X->world; r++) M.region[r] = X->peer[r];
    M.own = (unsigned long long*)X->own;
    M.bnd = D.bnd;
    M.hold = D.bnd_hold;
    M.base = W->bnd_base;
    M.last = X->last;
    M.nb = D.n_bnd;
    M.slot_bytes = sizeof(unsigned long long) * nbs;
    M.epoch0 = X->epoch;
    M.timeout_ns = 60ull * 1000000000ull;
    M.eps_fx = (unsigned long long)(S.eps * 4294967296.0);
    M.world = X->world;
    M.rank = X->rank;
    M.every = (int)std::max<int64_t>(1, local_rounds);
    M.sum = S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION;
    M.mark = scc_marks(W, S) != nullptr;
    int rc;
    if ((rc = launch_path(W, D, launch_algo(S), (int)std::min<int64_t>(max_rounds, 1 << 30), S, err, &M))) return rc;
    Counters c;
    if ((rc = read_counters(W, c, err))) return rc;
    X->epoch += c.mr_ex;
    *exchanges = (int64_t)c.mr_ex;
    if (c.mr_err) { err = "dg_run_fused: a peer did not arrive within 60 s"; return DG_ETIMEOUT; }
    *converged = c.mr_ex > 0 && c.mr_total == 0;
    return DG_OK;
}

int dev_run_end(DevWork* W, const DevLayout& D, RunState& S, std::string& err) {
    CK(cudaEventRecord(W->ev1));
    CK(cudaEventSynchronize(W->ev1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, W->ev0, W->ev1));
    int rc;
    if ((rc = S.algo == DG_SCC ? fold_counters(W, S, err) : collect_stats(W, S, err))) return rc;
    S.stats.time_ms = ms;
    return DG_OK;
}

int dev_normalize(void* buf, int64_t n, std::string& err) {
    double* d = nullptr;
    CK(cudaMalloc(&d, sizeof(double)));
    CK(cudaMemset(d, 0, sizeof(double)));
    sum_f_kernel<<<grid_1d(n), 256>>>((const float*)buf, n, d);
    scale_f_kernel<<<grid_1d(n), 256>>>((float*)buf, n, d);
    cudaError_t e = cudaGetLastError();
    cudaDeviceSynchronize();
    cudaFree(d);
    if (e != cudaSuccess) { err = cudaGetErrorString(e); return DG_ENOCUDA; }
    return DG_OK;
}

int dev_get_states(DevWork* W, const DevLayout& D, const RunState& S, void* out, int64_t n, int out_is_device,
                   std::string& err) {
    if (!W) { err = "no run state"; return DG_EINVAL; }
    void* dst = out;
    void* tmp = nullptr;
    if (!out_is_device) {  // device staging buffer kept in the work set (no cudaMalloc per call)
        int64_t bytes = 0;
        int rc;
        if (!W->out_stage && (rc = dalloc(&W->out_stage, (size_t)std::max<int64_t>(n, 1), bytes, err))) return rc;
        tmp = W->out_stage;
        dst = tmp;
    }
    const int g = grid_1d(n);
    if (S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION) {
        const unsigned long long* va = S.mode == DG_MODE_PATH ? W->vs_t : nullptr;
        CK(cudaMemset(W->dsum, 0, sizeof(double)));
        if (S.algo == DG_PAGERANK) sum_T_kernel<<<g, 256>>>(W->vs_f, va, n, W->dsum);
        out_pr_kernel<<<g, 256>>>(W->vs_f, va, D.new_id, n, W->dsum, (float*)dst,
                                  S.algo == DG_PAGERANK && !S.raw_states);
    } else if (S.algo == DG_SCC) {
        out_i_kernel<<<g, 256>>>(W->scc_label, D.new_id, n, (int32_t*)dst);
    } else {
        out_u_kernel<<<g, 256>>>(W->vs_u, D.new_id, n, (uint32_t*)dst);
    }
    CK(cudaGetLastError());
    if (tmp) {
        // D2H into a pinned staging buffer at full link speed, then a parallel
        // host copy into the caller's (pageable) buffer: a copy straight into
        // pageable memory runs at a fraction of the link (166 MB in 37 ms for
        // the Twitter-shaped graph)
        if (W->host_stage_n < n) {
            if (W->host_stage) cudaFreeHost(W->host_stage);
            W->host_stage = nullptr;
            W->host_stage_n = 0;
            if (cudaHostAlloc(&W->host_stage, 4 * (size_t)std::max<int64_t>(n, 1), cudaHostAllocDefault) == cudaSuccess)
                W->host_stage_n = n;
            else
                cudaGetLastError();
        }
        if (W->host_stage) {
            cudaError_t e = cudaMemcpy(W->host_stage, tmp, 4 * (size_t)n, cudaMemcpyDeviceToHost);
            if (e != cudaSuccess) { err = cudaGetErrorString(e); return DG_ENOCUDA; }
            const int64_t chunk = 1 << 20;
#pragma omp parallel for schedule(static)
            for (int64_t b = 0; b < (n + chunk - 1) / chunk; b++) {
                const int64_t lo = b * chunk, hi = std::min<int64_t>(n, lo + chunk);
                std::memcpy((uint32_t*)out + lo, (const uint32_t*)W->host_stage + lo, 4 * (size_t)(hi - lo));
            }
        } else {  // no pinned memory available: direct copy
            cudaError_t e = cudaMemcpy(out, tmp, 4 * (size_t)n, cudaMemcpyDeviceToHost);
            if (e != cudaSuccess) { err = cudaGetErrorString(e); return DG_ENOCUDA; }
        }
    } else {
        CK(cudaDeviceSynchronize());
    }
    return DG_OK;
}

}  // namespace dg
