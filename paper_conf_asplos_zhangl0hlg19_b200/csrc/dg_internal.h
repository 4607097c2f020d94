// Internal declarations shared by the host preprocessing (dg_host.cpp) and
// the CUDA kernels (dg_kernels.cu).  Not part of the public ABI.
#pragma once
#include <cstdint>
#include <functional>
#include <string>
#include <vector>

#include "../../include/digraph.h"

namespace dg {

// Path entry encoding in e_idx (uint32): internal vertex id in bits 0..29,
// bit 31 = first vertex of a path (head), bit 30 = last vertex (tail).
// Internal ids: the n_proxy highest-degree vertices are renumbered to
// [0, n_proxy) (shared-memory proxy vertices); every other
// vertex keeps its id unless it was displaced by a hub.
constexpr uint32_t kHead = 0x80000000u;
constexpr uint32_t kTail = 0x40000000u;
constexpr uint32_t kVMask = 0x3FFFFFFFu;

struct HostCSR {
    int64_t n = 0, m = 0;
    std::vector<int64_t> row_ptr;
    std::vector<int32_t> col, w;
    bool has_w = false;
    int32_t max_w = 1;  // largest edge weight (1 without weights)
    std::vector<int32_t> indeg, outdeg;
};

// Host copy of the built layout (one rank's share).
struct HostLayout {
    bool built = false;
    mutable int64_t hub_entries = -1;   // entries of vertices [0, n_proxy), counted on first request
    dg_path_params params{};
    // paths of this rank in priority order
    std::vector<int64_t> path_off;      // n_paths+1, into entries
    std::vector<int32_t> layer;         // per path
    std::vector<int64_t> scc;           // canonical dependency-SCC label per path
    std::vector<int64_t> merged_index;  // merge-order index per path
    std::vector<uint8_t> hot;           // per path
    // entries
    std::vector<uint32_t> e_idx;        // vertex | head | tail
    std::vector<int32_t> e_w;           // weight of the path edge INTO this entry (0 at heads)
    std::vector<int64_t> part_off;      // n_part+1
    // internal numbering and the CSR in internal ids (device copy for the
    // ablation, Adsorption weights and out-degrees)
    int64_t n_proxy = 0;
    std::vector<int32_t> new_id, orig;  // original -> internal, internal -> original
    std::vector<int64_t> prow_ptr;
    std::vector<int32_t> pcol, pw, poutdeg;
    std::vector<int64_t> srow_ptr;       // both directions (WCC ablation), built on first use
    std::vector<int32_t> scol;
    // multi-rank
    std::vector<int32_t> boundary;      // internal ids of vertices present on >1 rank (ascending)
    std::vector<uint64_t> bnd_hold;     // per boundary vertex: bit r set iff rank r's paths hold it
    std::vector<float> wsum;            // per vertex (internal ids): sum of out-edge weights (Adsorption)
    bool has_csr = true;                // prow_ptr/pcol/pw present (false: loaded from a layout file)
    // stats
    int64_t n_layers = 0, n_dep_sccs = 0, giant = 0, paths_before_merge = 0, n_hot = 0;
    double preprocess_ms = 0;
};

void build_layout(const HostCSR& g, const dg_path_params& p, HostLayout& L);
// One preprocessing pass for several ranks of a multi-rank layout: everything
// but the rank selection runs once; emit(rank, L) receives each rank's layout
// (L is reused between calls).
void build_layouts(const HostCSR& g, const dg_path_params& p, const std::vector<int>& ranks,
                   const std::function<void(int, HostLayout&)>& emit);
// Layout files (dg_save_layout / dg_load_layout): the layout without the CSR
// arrays, plus the graph's n, m, has_w and max_w.
int save_layout(const HostCSR& g, const HostLayout& L, const char* path, std::string& err);
int load_layout(HostCSR& g, HostLayout& L, const char* path, std::string& err);

// ---------------- device side ----------------
struct DevLayout {
    int64_t n = 0, m = 0, M = 0, n_part = 0, n_bnd = 0, max_part = 0;
    uint32_t* e_idx = nullptr;
    int32_t* e_w = nullptr;
    int64_t* part_off = nullptr;
    int32_t* bnd = nullptr;
    unsigned long long* bnd_hold = nullptr;  // holder ranks of each boundary vertex
    int32_t* new_id = nullptr;  // original -> internal
    int32_t* orig = nullptr;    // internal -> original
    int64_t n_proxy = 0;
    // CSR (for the vertex-centric ablation and per-vertex coefficients)
    int64_t* row_ptr = nullptr; int32_t* col = nullptr; int32_t* w = nullptr;
    int32_t* outdeg = nullptr;
    int64_t* srow_ptr = nullptr; int32_t* scol = nullptr;  // both directions (WCC ablation)
    int64_t bytes = 0;      // device bytes allocated
    int64_t h2d_bytes = 0;  // bytes copied host -> device since the last dg_upload
    bool csr_ok = false, ew_ok = false, sym_ok = false;  // lazily uploaded parts present
    std::vector<void*> pinned;  // host buffers page-locked with cudaHostRegister
};
void dev_unpin_all(DevLayout& D);

struct DevWork;  // defined in dg_kernels.cu

struct RunState {
    int algo = -1, mode = 0;
    int64_t source = 0;
    double eps = 0, param = 0;
    int64_t delta = 0;  // SSSP/BFS bucket width (reading R-DELTA), 0 = unbounded
    int64_t round = 0;
    bool raw_states = false;  // multi-rank: per-rank additive contributions, not normalised
    int scc_phase = -1;       // multi-rank SCC: 0 forward colouring, 1 backward marks, -1 between
    dg_run_stats stats{};
};

// Kernel-side entry points (dg_kernels.cu).  All return 0 or DG_E*.
int dev_select(int device, std::string& err);
int dev_upload_csr(DevLayout& D, const HostCSR& g, const HostLayout& L, std::string& err);
int dev_upload_layout(DevLayout& D, const HostLayout& L, std::string& err);
int dev_ensure_parts(DevLayout& D, const HostCSR& g, const HostLayout& L, bool need_csr, bool need_ew, bool need_sym,
                     std::string& err);
void dev_free_layout(DevLayout& D, bool csr_too);
int dev_set_vertex_params(DevWork*& W, const DevLayout& D, const double* p_inj, const double* p_cont,
                          const double* inj, const float* wsum, std::string& err);
int dev_run(DevWork*& W, const DevLayout& D, RunState& S, int64_t max_rounds, std::string& err);
int dev_run_begin(DevWork*& W, const DevLayout& D, RunState& S, std::string& err);
int dev_rounds(DevWork* W, const DevLayout& D, RunState& S, int64_t max_rounds, int64_t* active, std::string& err);
int dev_boundary_pack(DevWork* W, const DevLayout& D, RunState& S, void* buf, std::string& err);
int dev_boundary_unpack(DevWork* W, const DevLayout& D, RunState& S, const void* buf, int64_t* active, std::string& err);
int dev_run_end(DevWork* W, const DevLayout& D, RunState& S, std::string& err);
int dev_scc_phase(DevWork* W, const DevLayout& D, RunState& S, int phase, int64_t* active, std::string& err);
int dev_scc_assign(DevWork* W, const DevLayout& D, RunState& S, int64_t* remaining, std::string& err);
struct P2P;  // peer-memory boundary exchange (dg_kernels.cu)
int dev_p2p_alloc(P2P*& X, const DevLayout& D, int world, int rank, void* handle, std::string& err);
int dev_p2p_open(P2P* X, const void* handles, std::string& err);
void dev_p2p_free(P2P*& X);
int dev_boundary_exchange(DevWork* W, const DevLayout& D, RunState& S, P2P* X, int64_t* active, std::string& err);
int dev_run_fused(DevWork* W, const DevLayout& D, RunState& S, P2P* X, int64_t local_rounds, int64_t max_rounds,
                  int64_t* exchanges, int64_t* converged, std::string& err);
int dev_normalize(void* buf, int64_t n, std::string& err);
int dev_get_states(DevWork* W, const DevLayout& D, const RunState& S, void* out, int64_t n, int out_is_device,
                   std::string& err);
void dev_free_work(DevWork*& W);
void dev_layout_changed(DevWork* W);  // device layout re-uploaded: drop arrays derived from it

}  // namespace dg
