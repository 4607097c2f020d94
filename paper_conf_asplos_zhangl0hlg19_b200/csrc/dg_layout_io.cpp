// Layout files (dg_save_layout / dg_load_layout / dg_build_paths_shared):
// the preprocessing result of one rank -- PAPER.md sec. 3.2.1 "the graph is
// preprocessed on the CPU" then paths are "dispatched from the host to the
// GPUs" (lines 104-114, 176) -- so a multi-rank run preprocesses once and
// hands every rank its share instead of every rank repeating Algorithm 1 on
// the whole graph.  A file holds the graph's n, m, weight flag and largest
// weight plus every HostLayout array except the CSR in internal ids (needed
// only by the vertex-centric ablation).  Host byte order; a version tag
// rejects files of another layout revision.
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "dg_internal.h"

namespace dg {
namespace {

constexpr char kMagic[8] = {'D', 'G', 'L', 'A', 'Y', 'O', 'U', 'T'};
constexpr uint32_t kVersion = 3;

struct Header {
    char magic[8];
    uint32_t version, has_w;
    int64_t n, m;
    int32_t max_w, pad;
    dg_path_params params;
    int64_t n_proxy, n_layers, n_dep_sccs, giant, paths_before_merge, n_hot;
    double preprocess_ms;
};

struct File {
    FILE* f = nullptr;
    ~File() {
        if (f) std::fclose(f);
    }
};

template <typename T>
bool put(FILE* f, const std::vector<T>& v) {
    const uint64_t c = v.size();
    return std::fwrite(&c, sizeof c, 1, f) == 1 && (c == 0 || std::fwrite(v.data(), sizeof(T), c, f) == c);
}
template <typename T>
bool get(FILE* f, std::vector<T>& v, uint64_t max_count) {
    uint64_t c = 0;
    if (std::fread(&c, sizeof c, 1, f) != 1 || c > max_count) return false;
    v.resize(c);
    return c == 0 || std::fread(v.data(), sizeof(T), c, f) == c;
}

}  // namespace

int save_layout(const HostCSR& g, const HostLayout& L, const char* path, std::string& err) {
    File F;
    F.f = std::fopen(path, "wb");
    if (!F.f) { err = std::string("cannot open ") + path + " for writing"; return DG_EINVAL; }
    Header h{};
    std::memcpy(h.magic, kMagic, 8);
    h.version = kVersion;
    h.has_w = g.has_w;
    h.n = g.n; h.m = g.m; h.max_w = g.max_w;
    h.params = L.params;
    h.n_proxy = L.n_proxy; h.n_layers = L.n_layers; h.n_dep_sccs = L.n_dep_sccs; h.giant = L.giant;
    h.paths_before_merge = L.paths_before_merge; h.n_hot = L.n_hot; h.preprocess_ms = L.preprocess_ms;
    bool ok = std::fwrite(&h, sizeof h, 1, F.f) == 1;
    ok = ok && put(F.f, L.path_off) && put(F.f, L.layer) && put(F.f, L.scc) && put(F.f, L.merged_index) &&
         put(F.f, L.hot) && put(F.f, L.e_idx) && put(F.f, L.e_w) && put(F.f, L.part_off) && put(F.f, L.new_id) &&
         put(F.f, L.orig) && put(F.f, L.poutdeg) && put(F.f, L.boundary) && put(F.f, L.wsum) && put(F.f, L.bnd_hold);
    if (!ok) { err = std::string("write failed: ") + path; return DG_EINVAL; }
    return DG_OK;
}

int load_layout(HostCSR& g, HostLayout& L, const char* path, std::string& err) {
    File F;
    F.f = std::fopen(path, "rb");
    if (!F.f) { err = std::string("cannot open ") + path; return DG_EINVAL; }
    Header h{};
    if (std::fread(&h, sizeof h, 1, F.f) != 1 || std::memcmp(h.magic, kMagic, 8) != 0) {
        err = std::string(path) + ": not a DiGraph layout file";
        return DG_EINVAL;
    }
    if (h.version != kVersion) { err = std::string(path) + ": layout file version mismatch"; return DG_EINVAL; }
    if (h.n < 0 || h.n >= (int64_t)kVMask || h.m < 0) { err = std::string(path) + ": bad n or m"; return DG_EINVAL; }
    HostCSR c;
    HostLayout l;
    c.n = h.n; c.m = h.m; c.has_w = h.has_w != 0; c.max_w = h.max_w;
    l.params = h.params;
    l.n_proxy = h.n_proxy; l.n_layers = h.n_layers; l.n_dep_sccs = h.n_dep_sccs; l.giant = h.giant;
    l.paths_before_merge = h.paths_before_merge; l.n_hot = h.n_hot; l.preprocess_ms = h.preprocess_ms;
    const uint64_t big = (uint64_t)1 << 40, nv = (uint64_t)h.n;
    bool ok = get(F.f, l.path_off, big) && get(F.f, l.layer, big) && get(F.f, l.scc, big) &&
              get(F.f, l.merged_index, big) && get(F.f, l.hot, big) && get(F.f, l.e_idx, big) &&
              get(F.f, l.e_w, big) && get(F.f, l.part_off, big) && get(F.f, l.new_id, nv) && get(F.f, l.orig, nv) &&
              get(F.f, l.poutdeg, nv) && get(F.f, l.boundary, nv) && get(F.f, l.wsum, nv) &&
              get(F.f, l.bnd_hold, nv);
    ok = ok && l.new_id.size() == nv && l.orig.size() == nv && l.poutdeg.size() == nv && l.wsum.size() == nv &&
         !l.part_off.empty() && l.e_w.size() == l.e_idx.size() && (uint64_t)l.part_off.back() == l.e_idx.size() &&
         l.bnd_hold.size() == l.boundary.size();
    if (!ok) { err = std::string(path) + ": truncated or inconsistent layout file"; return DG_EINVAL; }
    l.has_csr = false;
    l.built = true;
    g = std::move(c);
    L = std::move(l);
    return DG_OK;
}

}  // namespace dg
