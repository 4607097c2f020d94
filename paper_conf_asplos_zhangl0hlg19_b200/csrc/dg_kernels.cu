// DiGraph hot path on sm_100a (B200): persistent path-propagation kernels,
// device-side convergence detection, the vertex-centric ablation and the
// multi-GPU boundary pack/unpack kernels.
//
// Path-based asynchronous execution (sec. 3.1, lines 94-96): the
// vertices of a path are handled in path order inside one round so a new
// state reaches the path's later vertices in the same round.  B200 mapping
// (DESIGN.md "Kernels"): one warp walks a partition (a run of whole paths,
// PAPER.md line 163 "the threads of a warp (assigned with a partition) read
// consecutive data") in windows of 128 path entries: lane l owns entries
// 4l..4l+3 (one 16-byte vector load of e_idx / e_w / S_val), gathers their
// master states, and the in-order walk along every path is computed exactly
// as a segmented warp scan (shuffles) of the per-entry transfer functions:
//   SSSP/BFS/WCC  x_i = min(a_i, x_{i-1} + w_i)        (min-plus, heads reset)
//   PR/Adsorption a_i = alpha_i + beta_i * a_{i-1}     (affine, heads reset)
// which is the sequential walk's result on the gathered snapshot.  Masters
// (V_val) change only through atomicMin / atomicAdd, and
// a changed master re-activates the partitions that read it (vertex ->
// partition maps).  All rounds run inside one cooperative persistent launch;
// partitions are dispatched from a device work list in priority order
// (layer, then hotness: PAPER.md lines 169, 192) and rounds end at a
// device-side active counter (north_star (4)).
#include <cooperative_groups.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstring>
#include <string>

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
constexpr int kPad = 256;  // entries of zero padding after the layout arrays

struct Counters {
    unsigned long long updates, edges, units, entries, pushes;
    int n_cur[2];
    unsigned int ticket[2];
    int round;  // global round number (stamps are round+1)
    int pad;
};

struct DevWork {
    int algo = -1, mode = -1;
    int grid_path = 0, grid_vertex = 0;
    uint2* vs_u = nullptr;      // {value, stamp}: SSSP/BFS dist, WCC label
    float4* vs_f = nullptr;     // {T, coef, sigma|delta, stamp}: PR / Adsorption
    float* e_coef = nullptr;    // Adsorption: coefficient of the path edge out of each entry
    float* ads_base = nullptr;  // Adsorption: p_inj * I per vertex
    float* ads_pcont = nullptr; // Adsorption: p_cont per vertex
    uint8_t* part_flag = nullptr;
    int32_t* plist[2] = {nullptr, nullptr};
    int32_t* vlist[2] = {nullptr, nullptr};
    int32_t* blockcnt = nullptr;
    Counters* ctr = nullptr;
    double* dsum = nullptr;
    int32_t* scc_color = nullptr;
    int32_t* scc_label = nullptr;
    uint8_t* scc_mark = nullptr;
    int32_t* remaining = nullptr;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr, kev0 = nullptr, kev1 = nullptr;
    bool have_params = false;
};

// ------------------------------------------------------------------ params
struct KParams {
    const uint32_t* e_idx;
    const int32_t* e_w;
    const int64_t* part_off;
    const int64_t* vsrc_ptr;
    const int32_t* vsrc;
    const int64_t* vdst_ptr;
    const int32_t* vdst;
    const int32_t* hpart;
    const int64_t* row_ptr;
    const int32_t* col;
    const int32_t* w;
    int64_t n_part, n;
    uint2* vs_u;
    float4* vs_f;
    const float* e_coef;
    uint8_t* part_flag;
    int32_t* plist0;
    int32_t* plist1;
    int32_t* vlist0;
    int32_t* vlist1;
    Counters* ctr;
    int32_t* blockcnt;
    // SCC
    int32_t* color;
    uint8_t* mark;
    const int32_t* scc_label;
    float eps;
    int max_rounds;
};

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
    asm volatile("ld.global.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                 : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
    return r;
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

// Warp-cooperative activation of the partitions listed for each vertex whose
// lane bit is set in `mask` (a master's new state must
// reach the paths holding its mirrors).
__device__ __forceinline__ void flag_partitions(uint32_t mask, int v, const int64_t* ptr, const int32_t* lst,
                                                uint8_t* flag) {
    const int lane = threadIdx.x & 31;
    while (mask) {
        int src = __ffs(mask) - 1;
        mask &= mask - 1;
        int vv = __shfl_sync(0xffffffffu, v, src);
        int64_t b = ptr[vv], e = ptr[vv + 1];
        for (int64_t j = b + lane; j < e; j += 32) flag[lst[j]] = 1;
    }
}

struct Acc {
    unsigned long long upd = 0, edges = 0, units = 0, entries = 0, pushes = 0;
};

// ------------------------------------------------------------------ path walks
// Min-plus walk (SSSP / BFS / WCC-forward).  MODE 0: SSSP weights, 1: BFS unit
// weights, 2: WCC (weight 0, both directions, both maps).
template <int MODE>
__device__ void walk_minplus(const KParams& P, int64_t beg, int64_t end, int round, Acc& acc) {
    const int lane = threadIdx.x & 31;
    uint32_t carry = INF;
    for (int64_t base = beg & ~(int64_t)3; base < end; base += 128) {
        const int64_t i0 = base + 4 * lane;
        uint4 code = make_uint4(kHead, kHead, kHead, kHead);
        int4 wv = make_int4(0, 0, 0, 0);
        if (i0 < end) {
            code = ld_stream_u4(P.e_idx + i0);
            if (MODE == 0) wv = ld_stream_i4(P.e_w + i0);
        }
        uint32_t a[4], wgt[4], vtx[4];
        bool hd[4], valid[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const int64_t i = i0 + k;
            valid[k] = i >= beg && i < end;
            uint32_t c = u4get(code, k);
            vtx[k] = c & kVMask;
            hd[k] = !valid[k] || (c & kHead);
            wgt[k] = MODE == 0 ? (uint32_t)i4get(wv, k) : (MODE == 1 ? 1u : 0u);
            a[k] = valid[k] ? P.vs_u[vtx[k]].x : INF;
        }
        // lane aggregate of f_k(x) = hd ? a : min(a, x + w)
        bool H = false;
        uint32_t A = INF, W = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            if (hd[k]) { H = true; A = a[k]; W = 0; }
            else { A = min(a[k], sat_add(A, wgt[k])); W = sat_add(W, wgt[k]); }
        }
        // warp inclusive scan (prefix composed before self)
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
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
        carry = __shfl_sync(0xffffffffu, cur, 31);
        if (MODE == 2) {
            // backward (suffix) min inside the window: x_i = min(a_i, x_{i+1}) until a tail
            bool T = false;
            uint32_t B = INF;
            bool tl[4];
#pragma unroll
            for (int k = 0; k < 4; k++) tl[k] = !valid[k] || (u4get(code, k) & kTail);
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
            bool Te = __shfl_down_sync(0xffffffffu, T, 1);
            uint32_t Be = __shfl_down_sync(0xffffffffu, B, 1);
            if (lane == 31) { Te = true; Be = INF; }
            uint32_t bc = Be;
            (void)Te;
#pragma unroll
            for (int k = 3; k >= 0; k--) {
                bc = tl[k] ? a[k] : min(a[k], bc);
                val[k] = min(val[k], bc);
            }
        }
        bool sig[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            sig[k] = false;
            if (valid[k]) {
                acc.entries++;
                if (!(u4get(code, k) & kHead)) acc.edges++;
                if (val[k] < a[k]) {
                    uint32_t old = atomicMin(&P.vs_u[vtx[k]].x, val[k]);
                    if (val[k] < old) {
                        acc.upd++;
                        sig[k] = atomicExch(&P.vs_u[vtx[k]].y, (uint32_t)(round + 1)) != (uint32_t)(round + 1);
                    }
                }
            }
        }
#pragma unroll
        for (int k = 0; k < 4; k++) {
            uint32_t m = __ballot_sync(0xffffffffu, sig[k]);
            if (m) {
                flag_partitions(m, (int)vtx[k], P.vsrc_ptr, P.vsrc, P.part_flag);
                if (MODE == 2) flag_partitions(m, (int)vtx[k], P.vdst_ptr, P.vdst, P.part_flag);
            }
        }
    }
}

// Accumulative walk (PageRank / Adsorption).
// Vertex state {r, g, delta, stamp}: r = accumulated value, delta = pending
// (fp32, small magnitudes -> no cancellation), g = per-vertex push factor
// (d/outdeg for PageRank, p_cont/W(u) for Adsorption).  Walking a path in
// order, entry i fires f_i = delta_i + p_i where delta_i is claimed from the
// master when >= eps (the per-vertex stop rule) and p_i = c_(i-1) * f_(i-1)
// is what its path predecessor just fired along the path edge -- used in the
// same round (Observation 1).  The in-window recurrence is
// the affine scan q_i = c_i * (delta_i + q_(i-1)).  A firing vertex adds f_i
// to r and pushes g*w*f_i to all its out-neighbours' deltas through the CSR
// (warp-cooperative, load-balanced); the amount p_i it already received
// in-register is debited from its own delta ("borrowed"), so mass is
// conserved exactly.  A delta crossing eps activates the vertex's home
// partition.
template <bool ADS>
__device__ void walk_delta(const KParams& P, int64_t beg, int64_t end, Acc& acc) {
    __shared__ int32_t s_v[kWarps][128];
    __shared__ float s_amt[kWarps][128];
    __shared__ int64_t s_row[kWarps][128];
    __shared__ int32_t s_off[kWarps][129];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const float eps = P.eps;
    for (int64_t base = beg & ~(int64_t)3; base < end; base += 128) {
        const int64_t i0 = base + 4 * lane;
        uint4 code = make_uint4(kHead | kTail, kHead | kTail, kHead | kTail, kHead | kTail);
        float4 c4 = make_float4(0.f, 0.f, 0.f, 0.f);
        if (i0 < end) {
            code = ld_stream_u4(P.e_idx + i0);
            if (ADS) c4 = ld_stream_f4(P.e_coef + i0);
        }
        float al[4], be[4], dl[4], gf[4];
        uint32_t vtx[4];
        bool hd[4], valid[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const int64_t i = i0 + k;
            valid[k] = i >= beg && i < end;
            uint32_t c = u4get(code, k);
            vtx[k] = c & kVMask;
            hd[k] = !valid[k] || (c & kHead);
            bool tl = !valid[k] || (c & kTail);
            float4 st = valid[k] ? P.vs_f[vtx[k]] : make_float4(0.f, 0.f, 0.f, 0.f);
            float d = 0.f;
            if (valid[k] && st.z >= eps) {
                d = atomicExch(&P.vs_f[vtx[k]].z, 0.f);
                if (d < 0.f) { atomicAdd(&P.vs_f[vtx[k]].z, d); d = 0.f; }
            }
            dl[k] = d;
            gf[k] = st.y;
            float cout = tl ? 0.f : (ADS ? f4get(c4, k) : st.y);
            al[k] = cout * d;
            be[k] = (tl || hd[k]) ? 0.f : cout;
        }
        float Al = 0.f, Be = 1.f;
#pragma unroll
        for (int k = 0; k < 4; k++) { Al = al[k] + be[k] * Al; Be = be[k] * Be; }
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            float Ap = __shfl_up_sync(0xffffffffu, Al, off);
            float Bp = __shfl_up_sync(0xffffffffu, Be, off);
            if (lane >= off) { Al = Al + Be * Ap; Be = Be * Bp; }
        }
        float prev = __shfl_up_sync(0xffffffffu, Al, 1);
        if (lane == 0) prev = 0.f;  // no carry across windows: earlier windows pushed through memory
        float f[4];
        bool fire[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            float pin = hd[k] ? 0.f : prev;
            prev = al[k] + be[k] * prev;
            f[k] = dl[k] + pin;
            fire[k] = valid[k] && f[k] > 0.f;
            if (valid[k]) acc.entries++;
            if (valid[k] && !hd[k]) acc.edges++;
            if (fire[k]) {
                atomicAdd(&P.vs_f[vtx[k]].x, f[k]);
                if (pin > 0.f) atomicAdd(&P.vs_f[vtx[k]].z, -pin);  // borrowed from the CSR push below
                acc.upd++;
            }
        }
        // gather the fired vertices of the window (<= 128) and expand their CSR rows
        int nit = 0;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            uint32_t m = __ballot_sync(0xffffffffu, fire[k]);
            if (fire[k]) {
                int pos = nit + __popc(m & ((1u << lane) - 1));
                s_v[wid][pos] = (int32_t)vtx[k];
                s_amt[wid][pos] = f[k] * gf[k];
            }
            nit += __popc(m);
        }
        __syncwarp();
        if (nit == 0) continue;
        int dsum = 0, dg4[4];
#pragma unroll
        for (int t = 0; t < 4; t++) {
            int it = lane * 4 + t;
            dg4[t] = 0;
            if (it < nit) {
                int v = s_v[wid][it];
                int64_t r0 = P.row_ptr[v];
                dg4[t] = (int)(P.row_ptr[v + 1] - r0);
                s_row[wid][it] = r0;
            }
            dsum += dg4[t];
        }
        int inc = dsum;
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            int y = __shfl_up_sync(0xffffffffu, inc, off);
            if (lane >= off) inc += y;
        }
        int run = inc - dsum;
#pragma unroll
        for (int t = 0; t < 4; t++) {
            int it = lane * 4 + t;
            if (it <= nit) s_off[wid][it] = run;
            run += dg4[t];
        }
        if (lane == 31 && nit == 128) s_off[wid][128] = inc;
        __syncwarp();
        const int total = s_off[wid][nit];
        for (int j = lane; j < total; j += 32) {
            int lo = 0, hi = nit - 1;  // owner: largest o with s_off[o] <= j
            while (lo < hi) {
                int mid = (lo + hi + 1) >> 1;
                if (s_off[wid][mid] <= j) lo = mid; else hi = mid - 1;
            }
            const int64_t e = s_row[wid][lo] + (j - s_off[wid][lo]);
            const int x = P.col[e];
            const float add = ADS ? s_amt[wid][lo] * (float)P.w[e] : s_amt[wid][lo];
            const float old = atomicAdd(&P.vs_f[x].z, add);
            if (old < eps && old + add >= eps) {
                const int hp = P.hpart[x];
                if (hp >= 0) P.part_flag[hp] = 1;  // -1: x lives on another rank (multi-GPU sync delivers it)
            }
            acc.pushes++;
        }
        __syncwarp();
    }
}

// SCC forward colouring: min colour along directed path edges restricted to
// unassigned vertices (scc_label < 0).  An assigned vertex breaks its paths.
__device__ void walk_scc_fwd(const KParams& P, int64_t beg, int64_t end, int round, Acc& acc) {
    const int lane = threadIdx.x & 31;
    uint32_t carry = INF;
    for (int64_t base = beg & ~(int64_t)3; base < end; base += 128) {
        const int64_t i0 = base + 4 * lane;
        uint4 code = make_uint4(kHead, kHead, kHead, kHead);
        if (i0 < end) code = ld_stream_u4(P.e_idx + i0);
        uint32_t a[4], vtx[4];
        bool hd[4], valid[4], live[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const int64_t i = i0 + k;
            valid[k] = i >= beg && i < end;
            uint32_t c = u4get(code, k);
            vtx[k] = c & kVMask;
            live[k] = valid[k] && P.scc_label[vtx[k]] < 0;
            hd[k] = !live[k] || (c & kHead);
            a[k] = live[k] ? P.vs_u[vtx[k]].x : INF;
        }
        bool H = false;
        uint32_t A = INF;
#pragma unroll
        for (int k = 0; k < 4; k++) {
            if (hd[k]) { H = true; A = a[k]; } else A = min(a[k], A);
        }
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
            bool Hp = __shfl_up_sync(0xffffffffu, H, off);
            uint32_t Ap = __shfl_up_sync(0xffffffffu, A, off);
            if (lane >= off && !H) { A = min(A, Ap); H = Hp; }
        }
        bool He = __shfl_up_sync(0xffffffffu, H, 1);
        uint32_t Ae = __shfl_up_sync(0xffffffffu, A, 1);
        if (lane == 0) { He = false; Ae = INF; }
        uint32_t cur = He ? Ae : min(Ae, carry);
        uint32_t val[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            cur = hd[k] ? a[k] : min(a[k], cur);
            val[k] = cur;
        }
        carry = __shfl_sync(0xffffffffu, cur, 31);
        bool sig[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            sig[k] = false;
            if (!live[k]) continue;
            acc.entries++;
            if (!(u4get(code, k) & kHead)) acc.edges++;
            if (val[k] < a[k]) {
                uint32_t old = atomicMin(&P.vs_u[vtx[k]].x, val[k]);
                if (val[k] < old) {
                    acc.upd++;
                    sig[k] = atomicExch(&P.vs_u[vtx[k]].y, (uint32_t)(round + 1)) != (uint32_t)(round + 1);
                }
            }
        }
#pragma unroll
        for (int k = 0; k < 4; k++) {
            uint32_t m = __ballot_sync(0xffffffffu, sig[k]);
            if (m) flag_partitions(m, (int)vtx[k], P.vsrc_ptr, P.vsrc, P.part_flag);
        }
    }
}

// SCC backward reachability inside a colour: walking each path backwards,
// mark_i |= mark_{i+1} when both are unassigned and share the colour.
// Windows are walked from the partition's end to its beginning so the
// suffix carry crosses windows.
__device__ void walk_scc_bwd(const KParams& P, int64_t beg, int64_t end, int round, Acc& acc) {
    const int lane = threadIdx.x & 31;
    bool carry = false;           // mark of the entry after the window
    uint32_t carry_col = INF;     // its colour (INF: none / tail boundary)
    const int64_t first = beg & ~(int64_t)3;
    int64_t nwin = (end - first + 127) / 128;
    for (int64_t wi = nwin - 1; wi >= 0; wi--) {
        const int64_t base = first + wi * 128;
        const int64_t i0 = base + 4 * lane;
        uint4 code = make_uint4(kTail, kTail, kTail, kTail);
        if (i0 < end) code = ld_stream_u4(P.e_idx + i0);
        uint32_t vtx[4], col[4];
        bool tl[4], valid[4], live[4], mk[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const int64_t i = i0 + k;
            valid[k] = i >= beg && i < end;
            uint32_t c = u4get(code, k);
            vtx[k] = c & kVMask;
            live[k] = valid[k] && P.scc_label[vtx[k]] < 0;
            tl[k] = !live[k] || (c & kTail);
            col[k] = live[k] ? P.vs_u[vtx[k]].x : INF;
            mk[k] = live[k] && P.mark[vtx[k]];
        }
        // transfer of element k on the mark coming from its successor x:
        //   m_k = mk_k | (x & eq_k),  eq_k = !tl_k && col_k == col_{k+1}
        // Represented as (or-term O, pass-flag Q): f(x) = O | (Q & x).
        // Need col_{k+1}: within lane, next element; for k=3 the next lane's k=0.
        uint32_t col_next_lane = __shfl_down_sync(0xffffffffu, col[0], 1);
        if (lane == 31) col_next_lane = carry_col;
        bool O[4], Q[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            uint32_t cn = k < 3 ? col[k + 1] : col_next_lane;
            bool eq = !tl[k] && col[k] == cn && cn != INF;
            O[k] = mk[k];
            Q[k] = eq;
        }
        // lane aggregate over elements 3..0 (suffix direction): F = f_0 o f_1 o f_2 o f_3
        bool AO = false, AQ = true;
#pragma unroll
        for (int k = 3; k >= 0; k--) { AO = O[k] | (Q[k] & AO); AQ = Q[k] & AQ; }
        // warp suffix scan (lanes above compose first)
#pragma unroll
        for (int off = 1; off < 32; off <<= 1) {
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
        // carry for the previous window: state of this window's first element
        bool first_m = __shfl_sync(0xffffffffu, newm[0], 0);
        uint32_t first_c = __shfl_sync(0xffffffffu, col[0], 0);
        carry = first_m;
        carry_col = first_c;
        bool sig[4];
#pragma unroll
        for (int k = 0; k < 4; k++) {
            sig[k] = false;
            if (!live[k]) continue;
            acc.entries++;
            if (!tl[k]) acc.edges++;
            if (newm[k] && !mk[k]) {
                // byte flag: plain store is idempotent
                P.mark[vtx[k]] = 1;
                acc.upd++;
                sig[k] = atomicExch(&P.vs_u[vtx[k]].y, (uint32_t)(round + 1)) != (uint32_t)(round + 1);
            }
        }
#pragma unroll
        for (int k = 0; k < 4; k++) {
            uint32_t m = __ballot_sync(0xffffffffu, sig[k]);
            if (m) flag_partitions(m, (int)vtx[k], P.vdst_ptr, P.vdst, P.part_flag);
        }
    }
}

// ------------------------------------------------------------------ round driver
// Ordered compaction of part_flag into the next work list (keeps priority
// order), executed by the whole cooperative grid.
__device__ void build_next_list(const KParams& P, int nxt, cg::grid_group& grid) {
    __shared__ int s_warp[kWarps];
    __shared__ int s_base;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int64_t slice = (P.n_part + gridDim.x - 1) / gridDim.x;
    const int64_t lo = min((int64_t)blockIdx.x * slice, P.n_part);
    const int64_t hi = min(lo + slice, P.n_part);
    int cnt = 0;
    for (int64_t q = lo + threadIdx.x; q < hi; q += blockDim.x) cnt += P.part_flag[q] != 0;
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if (lane == 0) s_warp[wid] = cnt;
    __syncthreads();
    if (threadIdx.x == 0) {
        int t = 0;
        for (int i = 0; i < kWarps; i++) t += s_warp[i];
        P.blockcnt[blockIdx.x] = t;
        if (blockIdx.x == 0) P.ctr->ticket[nxt] = 0;
    }
    grid.sync();
    if (threadIdx.x == 0) {
        int base = 0, total = 0;
        for (unsigned b = 0; b < gridDim.x; b++) {
            int c = P.blockcnt[b];
            if (b < blockIdx.x) base += c;
            total += c;
        }
        s_base = base;
        if (blockIdx.x == 0) P.ctr->n_cur[nxt] = total;
    }
    __syncthreads();
    int32_t* out = nxt ? P.plist1 : P.plist0;
    for (int64_t q0 = lo; q0 < hi; q0 += blockDim.x) {
        int64_t q = q0 + threadIdx.x;
        bool f = q < hi && P.part_flag[q] != 0;
        unsigned b = __ballot_sync(0xffffffffu, f);
        int pre = __popc(b & ((1u << lane) - 1));
        if (lane == 0) s_warp[wid] = __popc(b);
        __syncthreads();
        int wbase = 0;
        for (int i = 0; i < wid; i++) wbase += s_warp[i];
        if (f) {
            out[s_base + wbase + pre] = (int32_t)q;
            P.part_flag[q] = 0;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            int t = 0;
            for (int i = 0; i < kWarps; i++) t += s_warp[i];
            s_base += t;
        }
        __syncthreads();
    }
}

template <int ALGO>
__global__ void __launch_bounds__(kBlock) path_kernel(KParams P) {
    cg::grid_group grid = cg::this_grid();
    const int lane = threadIdx.x & 31;
    Acc acc;
    int r = 0;
    for (; r < P.max_rounds; r++) {
        const int round = P.ctr->round + r;  // ctr->round only changes after the kernel
        const int cur = round & 1;
        const int ncur = *((volatile int*)&P.ctr->n_cur[cur]);
        if (ncur == 0) break;
        const int32_t* list = cur ? P.plist1 : P.plist0;
        while (true) {
            unsigned t = 0;
            if (lane == 0) t = atomicAdd(&P.ctr->ticket[cur], 1u);
            t = __shfl_sync(0xffffffffu, t, 0);
            if (t >= (unsigned)ncur) break;
            const int q = list[t];
            const int64_t beg = P.part_off[q], end = P.part_off[q + 1];
            acc.units++;
            if (ALGO == DG_SSSP) walk_minplus<0>(P, beg, end, round, acc);
            else if (ALGO == DG_BFS) walk_minplus<1>(P, beg, end, round, acc);
            else if (ALGO == DG_WCC) walk_minplus<2>(P, beg, end, round, acc);
            else if (ALGO == DG_PAGERANK) walk_delta<false>(P, beg, end, acc);
            else if (ALGO == DG_ADSORPTION) walk_delta<true>(P, beg, end, acc);
            else if (ALGO == 100) walk_scc_fwd(P, beg, end, round, acc);
            else if (ALGO == 101) walk_scc_bwd(P, beg, end, round, acc);
        }
        grid.sync();
        build_next_list(P, cur ^ 1, grid);
        grid.sync();
    }
    // statistics (lane 0 of each warp)
    for (int off = 16; off; off >>= 1) {
        acc.upd += __shfl_xor_sync(0xffffffffu, acc.upd, off);
        acc.edges += __shfl_xor_sync(0xffffffffu, acc.edges, off);
        acc.entries += __shfl_xor_sync(0xffffffffu, acc.entries, off);
        acc.pushes += __shfl_xor_sync(0xffffffffu, acc.pushes, off);
    }
    if (lane == 0) {
        atomicAdd(&P.ctr->updates, acc.upd);
        atomicAdd(&P.ctr->edges, acc.edges);
        atomicAdd(&P.ctr->units, acc.units);
        atomicAdd(&P.ctr->entries, acc.entries);
        atomicAdd(&P.ctr->pushes, acc.pushes);
    }
    grid.sync();
    if (blockIdx.x == 0 && threadIdx.x == 0) P.ctr->round += r;
}

// ------------------------------------------------------------------ vertex-centric ablation
// Bulk-synchronous frontier kernel over the CSR (Gunrock-style baseline the
// paper compares against, sec. 2 "existing synchronous GPU-based
// methods"): every round each frontier vertex pushes along all its out-edges;
// warps load-balance the edges of 32 frontier vertices with a prefix sum.
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
        const int ncur = *((volatile int*)&P.ctr->n_cur[cur]);
        if (ncur == 0) break;
        const int32_t* list = cur ? P.vlist1 : P.vlist0;
        int32_t* out = nxt ? P.vlist1 : P.vlist0;
        while (true) {
            unsigned t = 0;
            if (lane == 0) t = atomicAdd(&P.ctr->ticket[cur], 32u);
            t = __shfl_sync(0xffffffffu, t, 0);
            if (t >= (unsigned)ncur) break;
            // claim up to 32 vertices
            int v = -1;
            int64_t deg = 0;
            if (t + lane < (unsigned)ncur) {
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
                    s_dist[wid][lane] = P.vs_u[v].x;
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
                    push = old < P.eps && old + a >= P.eps;
                } else {
                    uint32_t cand = sat_add(s_dist[wid][lo], ALGO == DG_BFS ? 1u : (uint32_t)P.w[e]);
                    if (cand < P.vs_u[x].x) {
                        uint32_t old = atomicMin(&P.vs_u[x].x, cand);
                        if (cand < old) { acc.upd++; push = true; }
                    }
                }
                if (push) {
                    unsigned* stp = ALGO == DG_PAGERANK ? reinterpret_cast<unsigned*>(&P.vs_f[x].w) : &P.vs_u[x].y;
                    if (atomicExch(stp, (unsigned)(round + 1)) != (unsigned)(round + 1)) {
                        int slot = atomicAdd(&P.ctr->n_cur[nxt], 1);
                        out[slot] = x;
                    }
                }
            }
            __syncwarp();
        }
        grid.sync();
        if (blockIdx.x == 0 && threadIdx.x == 0) { P.ctr->n_cur[cur] = 0; P.ctr->ticket[cur] = 0; }
        grid.sync();
    }
    for (int off = 16; off; off >>= 1) {
        acc.upd += __shfl_xor_sync(0xffffffffu, acc.upd, off);
        acc.edges += __shfl_xor_sync(0xffffffffu, acc.edges, off);
        acc.units += __shfl_xor_sync(0xffffffffu, acc.units, off);
        acc.pushes += __shfl_xor_sync(0xffffffffu, acc.pushes, off);
    }
    if (lane == 0) {
        atomicAdd(&P.ctr->updates, acc.upd);
        atomicAdd(&P.ctr->edges, acc.edges);
        atomicAdd(&P.ctr->units, acc.units);
        atomicAdd(&P.ctr->pushes, acc.pushes);
    }
    grid.sync();
    if (blockIdx.x == 0 && threadIdx.x == 0) P.ctr->round += r;
}

// ------------------------------------------------------------------ small kernels
__global__ void init_u_kernel(uint2* vs, int64_t n, int algo, int64_t source) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        uint32_t val = (algo == DG_WCC) ? (uint32_t)v : (v == source ? 0u : INF);
        vs[v] = make_uint2(val, 0u);
    }
}
// {r, g, delta, stamp}: r = 0, delta = 1-d (unnormalised PageRank, reading R-PR)
// With several ranks only the vertex's owner rank starts with the delta, so
// per-rank contributions add up (multi-GPU gather = sum).
__global__ void init_pr_kernel(float4* vs, const int32_t* outdeg, const uint8_t* vown, int64_t n, float d) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        float c = outdeg[v] > 0 ? d / (float)outdeg[v] : 0.f;
        vs[v] = make_float4(0.f, c, vown[v] ? 1.f - d : 0.f, 0.f);
    }
}
// Adsorption: r = 0, delta = p_inj * I, g = p_cont / W(u)
__global__ void init_ads_kernel(float4* vs, const float* base, const float* gfac, const uint8_t* vown, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        vs[v] = make_float4(0.f, gfac[v], vown[v] ? base[v] : 0.f, 0.f);
}
__global__ void gfac_kernel(float* pcont_to_g, const float* wsum, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        pcont_to_g[v] = wsum[v] > 0.f ? pcont_to_g[v] / wsum[v] : 0.f;
}
__global__ void fill_iota_kernel(int32_t* a, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        a[i] = (int32_t)i;
}
// Adsorption per-entry coefficient of the path edge out of entry i:
// p_cont(u) * w(u, next) / W(u), W(u) = sum of u's out-weights.
__global__ void ads_coef_kernel(float* e_coef, const uint32_t* e_idx, const int32_t* e_w, const float* pcont,
                                const float* wsum, int64_t M) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < M; i += (int64_t)gridDim.x * blockDim.x) {
        uint32_t c = e_idx[i];
        float x = 0.f;
        if (!(c & kTail)) {
            uint32_t u = c & kVMask;
            x = pcont[u] * (float)e_w[i + 1] / wsum[u];
        }
        e_coef[i] = x;
    }
}
__global__ void wsum_kernel(float* wsum, const int64_t* row_ptr, const int32_t* w, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        double s = 0;
        for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; e++) s += w ? (double)w[e] : 1.0;
        wsum[v] = (float)s;
    }
}
__global__ void sum_T_kernel(const float4* vs, int64_t n, double* out) {
    double s = 0;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        float4 x = vs[v];
        s += (double)x.x + (double)x.z;
    }
    for (int off = 16; off; off >>= 1) s += __shfl_xor_sync(0xffffffffu, s, off);
    if ((threadIdx.x & 31) == 0) atomicAdd(out, s);
}
__global__ void out_pr_kernel(const float4* vs, int64_t n, const double* sum, float* out, int normalize) {
    const double inv = normalize ? 1.0 / *sum : 1.0;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        float4 x = vs[v];
        out[v] = (float)(((double)x.x + (double)x.z) * inv);
    }
}
__global__ void out_u_kernel(const uint2* vs, int64_t n, uint32_t* out) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        out[v] = vs[v].x;
}
// Seed the work list with the partitions reading `source` (SSSP/BFS).
__global__ void seed_source_kernel(const int64_t* ptr, const int32_t* lst, int64_t source, int32_t* plist,
                                   Counters* ctr) {
    int64_t b = ptr[source], e = ptr[source + 1];
    for (int64_t j = b + threadIdx.x; j < e; j += blockDim.x) plist[j - b] = lst[j];
    if (threadIdx.x == 0) { ctr->n_cur[0] = (int)(e - b); ctr->n_cur[1] = 0; }
}

// ---- SCC helpers
__global__ void scc_init_kernel(uint2* vs, const int32_t* label, uint8_t* mark, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        vs[v] = make_uint2(label[v] < 0 ? (uint32_t)v : INF, 0u);
        mark[v] = 0;
    }
}
__global__ void scc_roots_kernel(const uint2* vs, const int32_t* label, uint8_t* mark, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        mark[v] = (label[v] < 0 && vs[v].x == (uint32_t)v) ? 1 : 0;
}
__global__ void scc_assign_kernel(const uint2* vs, int32_t* label, const uint8_t* mark, int64_t n, int32_t* remaining) {
    int cnt = 0;
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x) {
        if (label[v] < 0) {
            if (mark[v]) label[v] = (int32_t)vs[v].x;
            else cnt++;
        }
    }
    for (int off = 16; off; off >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, off);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(remaining, cnt);
}
// Seed the SCC backward phase: partitions holding a root as a non-head entry.
__global__ void scc_seed_bwd_kernel(const uint8_t* mark, const int32_t* label, const int64_t* ptr, const int32_t* lst,
                                    uint8_t* flag, int64_t n) {
    for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
        if (mark[v] && label[v] < 0)
            for (int64_t j = ptr[v]; j < ptr[v + 1]; j++) flag[lst[j]] = 1;
}

// ---- multi-GPU boundary exchange
__global__ void pack_min_kernel(const uint2* vs, const int32_t* bnd, int64_t nb, uint32_t* buf) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nb; k += (int64_t)gridDim.x * blockDim.x)
        buf[k] = vs[bnd[k]].x;
}
__global__ void unpack_min_kernel(uint2* vs, const int32_t* bnd, int64_t nb, const uint32_t* buf, int round,
                                  const int64_t* ptr, const int32_t* lst, const int64_t* ptr2, const int32_t* lst2,
                                  uint8_t* flag) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nb; k += (int64_t)gridDim.x * blockDim.x) {
        int v = bnd[k];
        if (buf[k] < vs[v].x) {
            vs[v].x = buf[k];
            vs[v].y = (uint32_t)(round + 1);
            for (int64_t j = ptr[v]; j < ptr[v + 1]; j++) flag[lst[j]] = 1;
            if (ptr2) for (int64_t j = ptr2[v]; j < ptr2[v + 1]; j++) flag[lst2[j]] = 1;
        }
    }
}
// SUM algorithms exchange the pending deltas of boundary vertices: every
// rank contributes its local delta, the owner rank receives the total
// ("each mirror always sends its new state to its master").
__global__ void pack_sum_kernel(const float4* vs, const int32_t* bnd, int64_t nb, float* buf) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nb; k += (int64_t)gridDim.x * blockDim.x)
        buf[k] = vs[bnd[k]].z;
}
__global__ void unpack_sum_kernel(float4* vs, const int32_t* bnd, const uint8_t* owner, int64_t nb, const float* buf,
                                  float eps, const int32_t* hpart, uint8_t* flag) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nb; k += (int64_t)gridDim.x * blockDim.x) {
        int v = bnd[k];
        float t = owner[k] ? buf[k] : 0.f;
        vs[v].z = t;
        if (t >= eps && hpart[v] >= 0) flag[hpart[v]] = 1;
    }
}
// single-block ordered compaction of part_flag (outside the persistent kernel)
__global__ void compact_flags_kernel(uint8_t* flag, int64_t n_part, int32_t* out, Counters* ctr, int slot) {
    __shared__ int s_warp[32];
    __shared__ int s_base;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
    if (threadIdx.x == 0) s_base = 0;
    __syncthreads();
    for (int64_t q0 = 0; q0 < n_part; q0 += blockDim.x) {
        int64_t q = q0 + threadIdx.x;
        bool f = q < n_part && flag[q] != 0;
        unsigned b = __ballot_sync(0xffffffffu, f);
        int pre = __popc(b & ((1u << lane) - 1));
        if (lane == 0) s_warp[wid] = __popc(b);
        __syncthreads();
        int wbase = 0;
        for (int i = 0; i < wid; i++) wbase += s_warp[i];
        if (f) { out[s_base + wbase + pre] = (int32_t)q; flag[q] = 0; }
        __syncthreads();
        if (threadIdx.x == 0) { int t = 0; for (int i = 0; i < nw; i++) t += s_warp[i]; s_base += t; }
        __syncthreads();
    }
    if (threadIdx.x == 0) { ctr->n_cur[slot] = s_base; ctr->ticket[slot] = 0; }
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
void dfree(T*& p) {
    if (p) cudaFree((void*)p);
    p = nullptr;
}
template <typename T>
int h2d(T* dst, const T* src, size_t count, std::string& err) {
    if (!count) return DG_OK;
    CK(cudaMemcpy(dst, src, sizeof(T) * count, cudaMemcpyHostToDevice));
    return DG_OK;
}
int grid_1d(int64_t n) {
    int64_t g = (n + 255) / 256;
    return (int)std::max<int64_t>(1, std::min<int64_t>(g, 148 * 16));
}

KParams make_params(const DevLayout& D, DevWork* W) {
    KParams P{};
    P.e_idx = D.e_idx; P.e_w = D.e_w; P.part_off = D.part_off;
    P.vsrc_ptr = D.vsrc_ptr; P.vsrc = D.vsrc; P.vdst_ptr = D.vdst_ptr; P.vdst = D.vdst; P.hpart = D.hpart;
    P.row_ptr = D.row_ptr; P.col = D.col; P.w = D.w;
    P.n_part = D.n_part; P.n = D.n;
    P.vs_u = W->vs_u; P.vs_f = W->vs_f; P.e_coef = W->e_coef;
    P.part_flag = W->part_flag; P.plist0 = W->plist[0]; P.plist1 = W->plist[1];
    P.vlist0 = W->vlist[0]; P.vlist1 = W->vlist[1];
    P.ctr = W->ctr; P.blockcnt = W->blockcnt;
    P.color = W->scc_color; P.mark = W->scc_mark; P.scc_label = W->scc_label;
    return P;
}

int ensure_work(DevWork*& W, const DevLayout& D, std::string& err) {
    if (W) return DG_OK;
    W = new DevWork();
    int64_t bytes = 0;
    int rc;
    if ((rc = dalloc(&W->vs_u, D.n, bytes, err))) return rc;
    if ((rc = dalloc(&W->vs_f, D.n, bytes, err))) return rc;
    if ((rc = dalloc(&W->part_flag, D.n_part + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->plist[0], std::max<int64_t>(D.n_part, D.n) + 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->plist[1], std::max<int64_t>(D.n_part, D.n) + 1, bytes, err))) return rc;
    W->vlist[0] = W->plist[0]; W->vlist[1] = W->plist[1];
    if ((rc = dalloc(&W->blockcnt, 148 * 64, bytes, err))) return rc;
    if ((rc = dalloc(&W->ctr, 1, bytes, err))) return rc;
    if ((rc = dalloc(&W->dsum, 1, bytes, err))) return rc;
    CK(cudaMemset(W->part_flag, 0, D.n_part + 1));
    CK(cudaEventCreate(&W->ev0));
    CK(cudaEventCreate(&W->ev1));
    CK(cudaEventCreate(&W->kev0));
    CK(cudaEventCreate(&W->kev1));
    return DG_OK;
}

int reset_counters(DevWork* W, std::string& err) {
    CK(cudaMemset(W->ctr, 0, sizeof(Counters)));
    return DG_OK;
}

int read_counters(DevWork* W, Counters& c, std::string& err) {
    CK(cudaMemcpy(&c, W->ctr, sizeof(Counters), cudaMemcpyDeviceToHost));
    return DG_OK;
}

// Launch the persistent path kernel for `rounds` rounds at most.
int launch_path(DevWork* W, const DevLayout& D, int algo_k, int rounds, float eps, RunState& S, std::string& err) {
    KParams P = make_params(D, W);
    P.eps = eps;
    P.max_rounds = rounds;
    void* args[] = {&P};
    void* fn = nullptr;
    switch (algo_k) {
        case DG_SSSP: fn = (void*)path_kernel<DG_SSSP>; break;
        case DG_BFS: fn = (void*)path_kernel<DG_BFS>; break;
        case DG_WCC: fn = (void*)path_kernel<DG_WCC>; break;
        case DG_PAGERANK: fn = (void*)path_kernel<DG_PAGERANK>; break;
        case DG_ADSORPTION: fn = (void*)path_kernel<DG_ADSORPTION>; break;
        case 100: fn = (void*)path_kernel<100>; break;
        case 101: fn = (void*)path_kernel<101>; break;
        default: err = "bad algo"; return DG_EINVAL;
    }
    int grid = 0;
    {
        int dev = 0, sms = 0, per = 0;
        CK(cudaGetDevice(&dev));
        CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, kBlock, 0));
        grid = sms * std::max(1, per);
    }
    CK(cudaEventRecord(W->kev0));
    CK(cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(kBlock), args, 0, 0));
    CK(cudaGetLastError());
    CK(cudaEventRecord(W->kev1));
    CK(cudaEventSynchronize(W->kev1));
    float kms = 0;
    CK(cudaEventElapsedTime(&kms, W->kev0, W->kev1));
    S.stats.kernel_ms += kms;
    S.stats.kernel_launches++;
    return DG_OK;
}

int launch_vertex(DevWork* W, const DevLayout& D, int algo, int rounds, float eps, RunState& S, std::string& err) {
    KParams P = make_params(D, W);
    P.eps = eps;
    P.max_rounds = rounds;
    void* args[] = {&P};
    void* fn = algo == DG_PAGERANK ? (void*)vertex_kernel<DG_PAGERANK>
             : algo == DG_BFS ? (void*)vertex_kernel<DG_BFS> : (void*)vertex_kernel<DG_SSSP>;
    int dev = 0, sms = 0, per = 0;
    CK(cudaGetDevice(&dev));
    CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, kBlock, 0));
    int grid = sms * std::max(1, per);
    CK(cudaEventRecord(W->kev0));
    CK(cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(kBlock), args, 0, 0));
    CK(cudaGetLastError());
    CK(cudaEventRecord(W->kev1));
    CK(cudaEventSynchronize(W->kev1));
    float kms = 0;
    CK(cudaEventElapsedTime(&kms, W->kev0, W->kev1));
    S.stats.kernel_ms += kms;
    S.stats.kernel_launches++;
    return DG_OK;
}

int init_states(DevWork* W, const DevLayout& D, RunState& S, std::string& err) {
    const int algo = S.algo;
    const int g = grid_1d(D.n);
    int rc;
    if ((rc = reset_counters(W, err))) return rc;
    if (S.mode == DG_MODE_VERTEX) {
        // frontier: the source (SSSP/BFS) or every vertex (PageRank)
        if (algo == DG_PAGERANK) {
            init_pr_kernel<<<g, 256>>>(W->vs_f, D.outdeg, D.vown, D.n, (float)S.param);
            fill_iota_kernel<<<g, 256>>>(W->vlist[0], D.n);
            int nn = (int)D.n;
            CK(cudaMemcpy(&W->ctr->n_cur[0], &nn, sizeof(int), cudaMemcpyHostToDevice));
            S.stats.kernel_launches += 2;
        } else {
            init_u_kernel<<<g, 256>>>(W->vs_u, D.n, algo, S.source);
            int32_t s = (int32_t)S.source;
            int one = 1;
            CK(cudaMemcpy(W->vlist[0], &s, sizeof(int32_t), cudaMemcpyHostToDevice));
            CK(cudaMemcpy(&W->ctr->n_cur[0], &one, sizeof(int), cudaMemcpyHostToDevice));
            S.stats.kernel_launches += 1;
        }
        CK(cudaGetLastError());
        return DG_OK;
    }
    CK(cudaMemsetAsync(W->part_flag, 0, D.n_part + 1));
    if (algo == DG_SSSP || algo == DG_BFS) {
        init_u_kernel<<<g, 256>>>(W->vs_u, D.n, algo, S.source);
        seed_source_kernel<<<1, 256>>>(D.vsrc_ptr, D.vsrc, S.source, W->plist[0], W->ctr);
        S.stats.kernel_launches += 2;
    } else if (algo == DG_WCC) {
        init_u_kernel<<<g, 256>>>(W->vs_u, D.n, algo, 0);
        fill_iota_kernel<<<grid_1d(D.n_part), 256>>>(W->plist[0], D.n_part);
        int np = (int)D.n_part;
        CK(cudaMemcpy(&W->ctr->n_cur[0], &np, sizeof(int), cudaMemcpyHostToDevice));
        S.stats.kernel_launches += 2;
    } else if (algo == DG_PAGERANK || algo == DG_ADSORPTION) {
        if (algo == DG_PAGERANK) init_pr_kernel<<<g, 256>>>(W->vs_f, D.outdeg, D.vown, D.n, (float)S.param);
        else init_ads_kernel<<<g, 256>>>(W->vs_f, W->ads_base, W->ads_pcont, D.vown, D.n);
        fill_iota_kernel<<<grid_1d(D.n_part), 256>>>(W->plist[0], D.n_part);
        int np = (int)D.n_part;
        CK(cudaMemcpy(&W->ctr->n_cur[0], &np, sizeof(int), cudaMemcpyHostToDevice));
        S.stats.kernel_launches += 2;
    }
    CK(cudaGetLastError());
    return DG_OK;
}

int collect_stats(DevWork* W, RunState& S, std::string& err) {
    Counters c;
    int rc;
    if ((rc = read_counters(W, c, err))) return rc;
    S.stats.rounds += c.round - (int)S.round;
    S.round = c.round;
    S.stats.vertex_updates = (int64_t)c.updates;
    S.stats.edges_processed = (int64_t)(c.edges + c.pushes);
    S.stats.units_processed = (int64_t)c.units;
    S.stats.entries_processed = (int64_t)c.entries;
    S.stats.csr_edges = (int64_t)c.pushes;
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
        if ((rc = dalloc(&W->scc_label, D.n, bytes, err))) return rc;
        if ((rc = dalloc(&W->scc_mark, D.n, bytes, err))) return rc;
        if ((rc = dalloc(&W->remaining, 1, bytes, err))) return rc;
    }
    const int g = grid_1d(D.n);
    CK(cudaMemset(W->scc_label, 0xff, sizeof(int32_t) * D.n));
    if ((rc = reset_counters(W, err))) return rc;
    int64_t total_rounds = 0;
    for (int64_t it = 0;; it++) {
        // forward colouring
        scc_init_kernel<<<g, 256>>>(W->vs_u, W->scc_label, W->scc_mark, D.n);
        CK(cudaMemset(W->part_flag, 0, D.n_part + 1));
        fill_iota_kernel<<<grid_1d(D.n_part), 256>>>(W->plist[0], D.n_part);
        Counters c0{};
        c0.n_cur[0] = (int)D.n_part;
        Counters cur;
        if ((rc = read_counters(W, cur, err))) return rc;
        c0.updates = cur.updates; c0.edges = cur.edges; c0.units = cur.units;
        c0.round = 0;
        CK(cudaMemcpy(W->ctr, &c0, sizeof(Counters), cudaMemcpyHostToDevice));
        S.stats.kernel_launches += 2;
        if ((rc = launch_path(W, D, 100, (int)max_rounds, 0.f, S, err))) return rc;
        Counters c1;
        if ((rc = read_counters(W, c1, err))) return rc;
        total_rounds += c1.round;
        // backward reachability from roots within colours
        scc_roots_kernel<<<g, 256>>>(W->vs_u, W->scc_label, W->scc_mark, D.n);
        CK(cudaMemset(W->part_flag, 0, D.n_part + 1));
        scc_seed_bwd_kernel<<<g, 256>>>(W->scc_mark, W->scc_label, D.vdst_ptr, D.vdst, W->part_flag, D.n);
        compact_flags_kernel<<<1, 1024>>>(W->part_flag, D.n_part, W->plist[0], W->ctr, 0);
        S.stats.kernel_launches += 3;
        // new stamps for the backward phase: reset the stamp half of vs_u and the round counter
        Counters c2;
        if ((rc = read_counters(W, c2, err))) return rc;
        c2.round = 0; c2.n_cur[1] = 0; c2.ticket[0] = c2.ticket[1] = 0;
        CK(cudaMemcpy(W->ctr, &c2, sizeof(Counters), cudaMemcpyHostToDevice));
        CK(cudaMemset2D(reinterpret_cast<char*>(W->vs_u) + 4, 8, 0, 4, D.n));
        if ((rc = launch_path(W, D, 101, (int)max_rounds, 0.f, S, err))) return rc;
        Counters c3;
        if ((rc = read_counters(W, c3, err))) return rc;
        total_rounds += c3.round;
        CK(cudaMemset(W->remaining, 0, sizeof(int32_t)));
        scc_assign_kernel<<<g, 256>>>(W->vs_u, W->scc_label, W->scc_mark, D.n, W->remaining);
        S.stats.kernel_launches += 1;
        int32_t rem = 0;
        CK(cudaMemcpy(&rem, W->remaining, sizeof(int32_t), cudaMemcpyDeviceToHost));
        S.stats.outer_iterations = it + 1;
        if (rem == 0) break;
        if (it > D.n) { err = "SCC colouring did not terminate"; return DG_ENOCONV; }
    }
    Counters cf;
    if ((rc = read_counters(W, cf, err))) return rc;
    S.stats.rounds = total_rounds;
    S.stats.vertex_updates = (int64_t)cf.updates;
    S.stats.edges_processed = (int64_t)cf.edges;
    S.stats.units_processed = (int64_t)cf.units;
    S.stats.entries_processed = (int64_t)cf.entries;
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

int dev_upload_csr(DevLayout& D, const HostCSR& g, std::string& err) {
    int dev_count = 0;
    if (cudaGetDeviceCount(&dev_count) != cudaSuccess || dev_count == 0) {
        err = "no CUDA device available (the DiGraph hot path has no CPU fallback)";
        return DG_ENOCUDA;
    }
    int rc;
    D.n = g.n; D.m = g.m;
    if ((rc = dalloc(&D.row_ptr, g.n + 1, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.col, g.m + kPad, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.outdeg, g.n, D.bytes, err))) return rc;
    if ((rc = h2d(D.row_ptr, g.row_ptr.data(), g.n + 1, err))) return rc;
    if ((rc = h2d(D.col, g.col.data(), g.m, err))) return rc;
    if ((rc = h2d(D.outdeg, g.outdeg.data(), g.n, err))) return rc;
    if (g.has_w) {
        if ((rc = dalloc(&D.w, g.m + kPad, D.bytes, err))) return rc;
        if ((rc = h2d(D.w, g.w.data(), g.m, err))) return rc;
    }
    return DG_OK;
}

int dev_upload_layout(DevLayout& D, const HostLayout& L, std::string& err) {
    int rc;
    D.M = (int64_t)L.e_idx.size();
    D.n_part = (int64_t)L.part_off.size() - 1;
    D.n_bnd = (int64_t)L.boundary.size();
    if ((rc = dalloc(&D.e_idx, D.M + kPad, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.e_w, D.M + kPad, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.part_off, D.n_part + 1, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.vsrc_ptr, D.n + 1, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.vsrc, L.vsrc.size(), D.bytes, err))) return rc;
    if ((rc = dalloc(&D.vdst_ptr, D.n + 1, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.vdst, L.vdst.size(), D.bytes, err))) return rc;
    if ((rc = dalloc(&D.bnd, D.n_bnd + 1, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.bnd_owner, D.n_bnd + 1, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.hpart, D.n + 1, D.bytes, err))) return rc;
    if ((rc = dalloc(&D.vown, D.n + 1, D.bytes, err))) return rc;
    if ((rc = h2d(D.bnd_owner, L.bnd_owner.data(), D.n_bnd, err))) return rc;
    if ((rc = h2d(D.hpart, L.hpart.data(), D.n, err))) return rc;
    if ((rc = h2d(D.vown, L.vown.data(), D.n, err))) return rc;
    CK(cudaMemset(D.e_idx + D.M, 0, sizeof(uint32_t) * kPad));
    CK(cudaMemset(D.e_w + D.M, 0, sizeof(int32_t) * kPad));
    if ((rc = h2d(D.e_idx, L.e_idx.data(), D.M, err))) return rc;
    if ((rc = h2d(D.e_w, L.e_w.data(), D.M, err))) return rc;
    if ((rc = h2d(D.part_off, L.part_off.data(), D.n_part + 1, err))) return rc;
    if ((rc = h2d(D.vsrc_ptr, L.vsrc_ptr.data(), D.n + 1, err))) return rc;
    if ((rc = h2d(D.vsrc, L.vsrc.data(), L.vsrc.size(), err))) return rc;
    if ((rc = h2d(D.vdst_ptr, L.vdst_ptr.data(), D.n + 1, err))) return rc;
    if ((rc = h2d(D.vdst, L.vdst.data(), L.vdst.size(), err))) return rc;
    if ((rc = h2d(D.bnd, L.boundary.data(), D.n_bnd, err))) return rc;
    CK(cudaDeviceSynchronize());
    return DG_OK;
}

void dev_free_layout(DevLayout& D, bool csr_too) {
    dfree(D.e_idx); dfree(D.e_w); dfree(D.part_off);
    dfree(D.vsrc_ptr); dfree(D.vsrc); dfree(D.vdst_ptr); dfree(D.vdst); dfree(D.bnd);
    dfree(D.bnd_owner); dfree(D.hpart); dfree(D.vown);
    if (csr_too) { dfree(D.row_ptr); dfree(D.col); dfree(D.w); dfree(D.outdeg); }
    D.bytes = 0;
    D.M = D.n_part = D.n_bnd = 0;
}

void dev_free_work(DevWork*& W) {
    if (!W) return;
    dfree(W->vs_u); dfree(W->vs_f); dfree(W->e_coef); dfree(W->ads_base); dfree(W->ads_pcont);
    dfree(W->part_flag); dfree(W->plist[0]); dfree(W->plist[1]); dfree(W->blockcnt); dfree(W->ctr);
    dfree(W->dsum); dfree(W->scc_color); dfree(W->scc_label); dfree(W->scc_mark);
    dfree(W->remaining);
    if (W->ev0) cudaEventDestroy(W->ev0);
    if (W->ev1) cudaEventDestroy(W->ev1);
    if (W->kev0) cudaEventDestroy(W->kev0);
    if (W->kev1) cudaEventDestroy(W->kev1);
    delete W;
    W = nullptr;
}

int dev_set_vertex_params(DevWork*& W, const DevLayout& D, const double* p_inj, const double* p_cont,
                          const double* inj, std::string& err) {
    int rc;
    if ((rc = ensure_work(W, D, err))) return rc;
    int64_t bytes = 0;
    if (!W->ads_base) {
        if ((rc = dalloc(&W->ads_base, D.n, bytes, err))) return rc;
        if ((rc = dalloc(&W->ads_pcont, D.n, bytes, err))) return rc;
        if ((rc = dalloc(&W->e_coef, D.M + kPad, bytes, err))) return rc;
    }
    std::vector<float> base(D.n), pc(D.n);
    for (int64_t v = 0; v < D.n; v++) { base[v] = (float)(p_inj[v] * inj[v]); pc[v] = (float)p_cont[v]; }
    if ((rc = h2d(W->ads_base, base.data(), D.n, err))) return rc;
    if ((rc = h2d(W->ads_pcont, pc.data(), D.n, err))) return rc;
    float* wsum = nullptr;
    if ((rc = dalloc(&wsum, D.n, bytes, err))) return rc;
    wsum_kernel<<<grid_1d(D.n), 256>>>(wsum, D.row_ptr, D.w, D.n);
    CK(cudaMemset(W->e_coef, 0, sizeof(float) * (D.M + kPad)));
    if (D.w) {
        ads_coef_kernel<<<grid_1d(D.M), 256>>>(W->e_coef, D.e_idx, D.e_w, W->ads_pcont, wsum, D.M);
        gfac_kernel<<<grid_1d(D.n), 256>>>(W->ads_pcont, wsum, D.n);
    } else {
        err = "Adsorption needs edge weights (load the CSR with weights)";
        cudaFree(wsum);
        return DG_EINVAL;
    }
    CK(cudaGetLastError());
    CK(cudaDeviceSynchronize());
    cudaFree(wsum);
    W->have_params = true;
    return DG_OK;
}

int dev_run(DevWork*& W, const DevLayout& D, RunState& S, int64_t max_rounds, std::string& err) {
    int rc;
    if ((rc = ensure_work(W, D, err))) return rc;
    if (S.algo == DG_ADSORPTION && !W->have_params) {
        err = "Adsorption needs dg_set_vertex_params first";
        return DG_EINVAL;
    }
    if (S.mode == DG_MODE_VERTEX && !D.row_ptr) { err = "CSR not on device"; return DG_EINVAL; }
    CK(cudaEventRecord(W->ev0));
    if (S.algo == DG_SCC) {
        if ((rc = run_scc(W, D, S, max_rounds, err))) return rc;
    } else {
        if ((rc = init_states(W, D, S, err))) return rc;
        const int rounds = (int)std::min<int64_t>(max_rounds, 1 << 30);
        if (S.mode == DG_MODE_VERTEX) rc = launch_vertex(W, D, S.algo, rounds, (float)S.eps, S, err);
        else rc = launch_path(W, D, S.algo, rounds, (float)S.eps, S, err);
        if (rc) return rc;
    }
    CK(cudaEventRecord(W->ev1));
    CK(cudaEventSynchronize(W->ev1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, W->ev0, W->ev1));
    if (S.algo != DG_SCC) {
        if ((rc = collect_stats(W, S, err))) return rc;
        Counters c;
        if ((rc = read_counters(W, c, err))) return rc;
        if (c.n_cur[c.round & 1] != 0) {
            S.stats.time_ms = ms;
            err = "max_rounds reached before convergence";
            return DG_ENOCONV;
        }
    }
    S.stats.time_ms = ms;
    return DG_OK;
}

int dev_run_begin(DevWork*& W, const DevLayout& D, RunState& S, std::string& err) {
    int rc;
    if ((rc = ensure_work(W, D, err))) return rc;
    if (S.algo == DG_ADSORPTION && !W->have_params) { err = "Adsorption needs dg_set_vertex_params first"; return DG_EINVAL; }
    if ((rc = init_states(W, D, S, err))) return rc;
    CK(cudaGetLastError());
    CK(cudaEventRecord(W->ev0));
    return DG_OK;
}

int dev_rounds(DevWork* W, const DevLayout& D, RunState& S, int64_t max_rounds, int64_t* active, std::string& err) {
    int rc;
    if ((rc = launch_path(W, D, S.algo, (int)std::min<int64_t>(max_rounds, 1 << 30), (float)S.eps, S, err))) return rc;
    Counters c;
    if ((rc = read_counters(W, c, err))) return rc;
    *active = c.n_cur[c.round & 1];
    return DG_OK;
}

int dev_boundary_pack(DevWork* W, const DevLayout& D, RunState& S, void* buf, std::string& err) {
    if (!D.n_bnd) return DG_OK;
    if (S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION)
        pack_sum_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_f, D.bnd, D.n_bnd, (float*)buf);
    else
        pack_min_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_u, D.bnd, D.n_bnd, (uint32_t*)buf);
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
    const int round = c.round;  // stamps of the next local round
    if (D.n_bnd) {
        if (S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION)
            unpack_sum_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_f, D.bnd, D.bnd_owner, D.n_bnd, (const float*)buf,
                                                         (float)S.eps, D.hpart, W->part_flag);
        else
            unpack_min_kernel<<<grid_1d(D.n_bnd), 256>>>(W->vs_u, D.bnd, D.n_bnd, (const uint32_t*)buf, round,
                                                         D.vsrc_ptr, D.vsrc,
                                                         S.algo == DG_WCC ? D.vdst_ptr : nullptr,
                                                         S.algo == DG_WCC ? D.vdst : nullptr, W->part_flag);
        S.stats.kernel_launches++;
    }
    // merge the flags into the current work list (ordered)
    compact_flags_kernel<<<1, 1024>>>(W->part_flag, D.n_part, W->plist[round & 1], W->ctr, round & 1);
    S.stats.kernel_launches++;
    CK(cudaGetLastError());
    if ((rc = read_counters(W, c, err))) return rc;
    *active = c.n_cur[round & 1];
    return DG_OK;
}

int dev_run_end(DevWork* W, const DevLayout& D, RunState& S, std::string& err) {
    CK(cudaEventRecord(W->ev1));
    CK(cudaEventSynchronize(W->ev1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, W->ev0, W->ev1));
    int rc;
    if ((rc = collect_stats(W, S, err))) return rc;
    S.stats.time_ms = ms;
    return DG_OK;
}

int dev_get_states(DevWork* W, const DevLayout& D, const RunState& S, void* out, int64_t n, int out_is_device,
                   std::string& err) {
    if (!W) { err = "no run state"; return DG_EINVAL; }
    void* dst = out;
    void* tmp = nullptr;
    if (!out_is_device) {
        CK(cudaMalloc(&tmp, 4 * (size_t)std::max<int64_t>(n, 1)));
        dst = tmp;
    }
    const int g = grid_1d(n);
    if (S.algo == DG_PAGERANK || S.algo == DG_ADSORPTION) {
        CK(cudaMemset(W->dsum, 0, sizeof(double)));
        if (S.algo == DG_PAGERANK) sum_T_kernel<<<g, 256>>>(W->vs_f, n, W->dsum);
        out_pr_kernel<<<g, 256>>>(W->vs_f, n, W->dsum, (float*)dst, S.algo == DG_PAGERANK);
    } else if (S.algo == DG_SCC) {
        CK(cudaMemcpy(dst, W->scc_label, 4 * (size_t)n, cudaMemcpyDeviceToDevice));
    } else {
        out_u_kernel<<<g, 256>>>(W->vs_u, n, (uint32_t*)dst);
    }
    CK(cudaGetLastError());
    if (tmp) {
        cudaError_t e = cudaMemcpy(out, tmp, 4 * (size_t)n, cudaMemcpyDeviceToHost);
        cudaFree(tmp);
        if (e != cudaSuccess) { err = cudaGetErrorString(e); return DG_ENOCUDA; }
    } else {
        CK(cudaDeviceSynchronize());
    }
    return DG_OK;
}

}  // namespace dg
