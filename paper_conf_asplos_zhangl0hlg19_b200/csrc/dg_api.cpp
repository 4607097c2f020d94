// C ABI of libdigraph.so (include/digraph.h): argument checking, lifecycle
// and dispatch to the host preprocessing (dg_preprocess.cpp) and the CUDA
// kernels (dg_kernels.cu).  No computation step of dg_run happens here.
#include <algorithm>
#include <cstring>
#include <vector>
#include <exception>
#include <new>
#include <string>

#include "dg_internal.h"

struct dg_graph {
    int device = 0;
    dg::HostCSR csr;
    dg::HostLayout layout;
    dg::DevLayout dev;
    dg::DevWork* work = nullptr;
    dg::P2P* p2p = nullptr;  // peer-memory exchange region (dg_p2p_alloc)
    dg::RunState run;
    bool loaded = false;
    bool uploaded = false;
    bool ran = false;
    bool multi_active = false;
};

namespace {
thread_local std::string g_err;

int fail(int code, const std::string& msg) {
    g_err = msg;
    return code;
}
}  // namespace

static int select_dev(dg_graph* g);

extern "C" {

const char* dg_last_error(void) { return g_err.c_str(); }

void dg_default_params(dg_path_params* p) {
    if (!p) return;
    p->d_max = 16;
    p->l_merge = 64;
    p->n_sub = 64;
    p->order = 0;
    p->hot_factor = 2.0f;
    p->part_entries = 0;
    p->rank = 0;
    p->world = 1;
    p->merge_rule = 1;
    p->n_proxy = 8192;
    p->placement = 1;
}

int dg_create(dg_graph** out, int device) {
    if (!out) return fail(DG_EINVAL, "dg_create: out is NULL");
    try {
        *out = new dg_graph();
        (*out)->device = device;
    } catch (const std::bad_alloc&) {
        return fail(DG_ENOMEM, "dg_create: out of host memory");
    }
    return DG_OK;
}

void dg_destroy(dg_graph* g) {
    if (!g) return;
    dg::dev_p2p_free(g->p2p);
    dg::dev_free_work(g->work);
    dg::dev_free_layout(g->dev, true);
    dg::dev_unpin_all(g->dev);
    delete g;
}

int dg_load_csr(dg_graph* g, int64_t n, int64_t m, const int64_t* row_ptr, const int32_t* col,
                const int32_t* weight) {
    if (!g) return fail(DG_EINVAL, "dg_load_csr: graph is NULL");
    if (n < 0 || n >= (int64_t)dg::kVMask || m < 0) return fail(DG_EINVAL, "dg_load_csr: bad n or m");
    if (!row_ptr || (m > 0 && !col)) return fail(DG_EINVAL, "dg_load_csr: NULL row_ptr/col");
    if (row_ptr[0] != 0 || row_ptr[n] != m) return fail(DG_EINVAL, "dg_load_csr: row_ptr[0] != 0 or row_ptr[n] != m");
    // validate into a local CSR and swap it in only on success: a failed load
    // leaves the handle (previous graph, layout and device state) untouched
    dg::HostCSR c;
    try {
        c.n = n; c.m = m;
        c.row_ptr.assign(row_ptr, row_ptr + n + 1);
        c.col.assign(col, col + m);
        c.has_w = weight != nullptr;
        if (weight) c.w.assign(weight, weight + m);
        c.max_w = 1;
        if (weight)
            for (int64_t e = 0; e < m; e++) c.max_w = std::max(c.max_w, weight[e]);
        c.indeg.assign(n, 0); c.outdeg.assign(n, 0);
        for (int64_t v = 0; v < n; v++) {
            if (row_ptr[v + 1] < row_ptr[v]) return fail(DG_EINVAL, "dg_load_csr: row_ptr decreasing");
            c.outdeg[v] = (int32_t)(row_ptr[v + 1] - row_ptr[v]);
        }
        for (int64_t k = 0; k < m; k++) {
            if (col[k] < 0 || col[k] >= n) return fail(DG_EINVAL, "dg_load_csr: column out of range");
            if (weight && weight[k] < 0) return fail(DG_EINVAL, "dg_load_csr: negative weight");
            c.indeg[col[k]]++;
        }
    } catch (const std::bad_alloc&) {
        return fail(DG_ENOMEM, "dg_load_csr: out of host memory");
    }
    // the old device state goes first: its host buffers are page-locked
    dg::dev_p2p_free(g->p2p);
    dg::dev_free_work(g->work);
    dg::dev_free_layout(g->dev, true);
    dg::dev_unpin_all(g->dev);
    g->csr = std::move(c);
    g->layout = dg::HostLayout();
    g->loaded = true;
    g->uploaded = false;
    g->ran = false;
    return DG_OK;
}

static int check_params(const dg_path_params& q) {
    if (q.d_max < 1 || q.n_sub < 1 || q.part_entries < 0 || q.world < 1 || q.world > 64 ||
        q.rank < 0 || q.rank >= q.world || q.l_merge < 0 || q.merge_rule < 0 || q.merge_rule > 1 ||
        q.n_proxy < 0 || q.n_proxy > 16384 || q.placement < 0 || q.placement > 1)
        return fail(DG_EINVAL, "dg_build_paths: bad parameters");
    return DG_OK;
}

int dg_build_paths(dg_graph* g, const dg_path_params* p) {
    if (!g || !g->loaded) return fail(DG_EINVAL, "dg_build_paths: no graph loaded");
    if (g->csr.row_ptr.empty())
        return fail(DG_EINVAL, "dg_build_paths: the graph came from a layout file (no CSR); use dg_load_csr");
    dg_path_params q;
    dg_default_params(&q);
    if (p) q = *p;
    if (int rc0 = check_params(q)) return rc0;
    dg::dev_p2p_free(g->p2p);
    dg::dev_free_work(g->work);
    dg::dev_free_layout(g->dev, true);
    dg::dev_unpin_all(g->dev);
    g->uploaded = false;
    try {
        dg::build_layout(g->csr, q, g->layout);
    } catch (const std::bad_alloc&) {
        return fail(DG_ENOMEM, "dg_build_paths: out of host memory");
    } catch (const std::exception& e) {
        return fail(DG_EINVAL, std::string("dg_build_paths: ") + e.what());
    }
    dg::dev_p2p_free(g->p2p);
    dg::dev_free_work(g->work);
    dg::dev_free_layout(g->dev, true);
    g->uploaded = false;
    g->ran = false;
    return DG_OK;
}

int dg_upload(dg_graph* g) {
    if (!g || !g->layout.built) return fail(DG_EINVAL, "dg_upload: no layout built");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    // a re-upload of the same layout copies into the existing device buffers
    // (and keeps the work buffers); a new layout was freed by dg_build_paths
    int rc = dg::dev_upload_csr(g->dev, g->csr, g->layout, err);
    if (!rc) rc = dg::dev_upload_layout(g->dev, g->layout, err);
    if (rc) { dg::dev_free_layout(g->dev, true); return fail(rc, err); }
    dg::dev_layout_changed(g->work);
    g->uploaded = true;
    g->ran = false;
    return DG_OK;
}

int dg_build_paths_shared(dg_graph* g, const dg_path_params* p, const char* prefix) {
    if (!g || !g->loaded || !p || !prefix) return fail(DG_EINVAL, "dg_build_paths_shared: no graph loaded or NULL argument");
    if (g->csr.row_ptr.empty())
        return fail(DG_EINVAL, "dg_build_paths_shared: the graph came from a layout file (no CSR)");
    if (int rc0 = check_params(*p)) return rc0;
    dg::dev_p2p_free(g->p2p);
    dg::dev_free_work(g->work);
    dg::dev_free_layout(g->dev, true);
    dg::dev_unpin_all(g->dev);
    g->uploaded = false;
    g->ran = false;
    g->layout = dg::HostLayout();
    std::vector<int> ranks;
    for (int r = 0; r < p->world; r++) ranks.push_back(r);
    std::string err;
    int rc = DG_OK;
    try {
        // ONE preprocessing pass emits every rank's share; this handle keeps its own
        dg::build_layouts(g->csr, *p, ranks, [&](int r, dg::HostLayout& L) {
            if (!rc) rc = dg::save_layout(g->csr, L, (std::string(prefix) + "." + std::to_string(r)).c_str(), err);
            if (r == p->rank) g->layout = L;
        });
    } catch (const std::bad_alloc&) {
        g->layout = dg::HostLayout();
        return fail(DG_ENOMEM, "dg_build_paths_shared: out of host memory");
    } catch (const std::exception& e) {
        g->layout = dg::HostLayout();
        return fail(DG_EINVAL, std::string("dg_build_paths_shared: ") + e.what());
    }
    if (rc) {
        g->layout = dg::HostLayout();
        return fail(rc, "dg_build_paths_shared: " + err);
    }
    return DG_OK;
}

int dg_save_layout(const dg_graph* g, const char* path) {
    if (!g || !g->layout.built || !path) return fail(DG_EINVAL, "dg_save_layout: no layout built or NULL path");
    std::string err;
    const int rc = dg::save_layout(g->csr, g->layout, path, err);
    return rc ? fail(rc, "dg_save_layout: " + err) : DG_OK;
}

int dg_load_layout(dg_graph* g, const char* path) {
    if (!g || !path) return fail(DG_EINVAL, "dg_load_layout: NULL argument");
    dg::HostCSR c;
    dg::HostLayout L;
    std::string err;
    int rc;
    try {
        rc = dg::load_layout(c, L, path, err);
    } catch (const std::bad_alloc&) {
        return fail(DG_ENOMEM, "dg_load_layout: out of host memory");
    }
    if (rc) return fail(rc, "dg_load_layout: " + err);  // the handle is unchanged
    dg::dev_p2p_free(g->p2p);
    dg::dev_free_work(g->work);
    dg::dev_free_layout(g->dev, true);
    dg::dev_unpin_all(g->dev);
    g->csr = std::move(c);
    g->layout = std::move(L);
    g->loaded = true;
    g->uploaded = false;
    g->ran = false;
    return DG_OK;
}

static int ensure_uploaded(dg_graph* g) {
    return g->uploaded ? DG_OK : dg_upload(g);
}

// The CSR of both edge directions (internal ids), for the WCC ablation:
// vertex x lists its out-neighbours, then its in-neighbours.
static void build_sym_csr(dg::HostLayout& L, int64_t n) {
    if (!L.srow_ptr.empty()) return;
    std::vector<int64_t> rp(n + 1, 0);
    for (int64_t u = 0; u < n; u++) {
        rp[u + 1] += L.prow_ptr[u + 1] - L.prow_ptr[u];
        for (int64_t e = L.prow_ptr[u]; e < L.prow_ptr[u + 1]; e++) rp[L.pcol[e] + 1]++;
    }
    for (int64_t u = 0; u < n; u++) rp[u + 1] += rp[u];
    std::vector<int32_t> col(rp[n]);
    std::vector<int64_t> cur(rp.begin(), rp.end() - 1);
    for (int64_t u = 0; u < n; u++)
        for (int64_t e = L.prow_ptr[u]; e < L.prow_ptr[u + 1]; e++) col[cur[u]++] = L.pcol[e];
    for (int64_t u = 0; u < n; u++)
        for (int64_t e = L.prow_ptr[u]; e < L.prow_ptr[u + 1]; e++) col[cur[L.pcol[e]]++] = (int32_t)u;
    L.srow_ptr.swap(rp);
    L.scol.swap(col);
}

// the parts of the device layout an algorithm reads beyond the path entries
static int ensure_parts(dg_graph* g, int algo, int mode) {
    const bool need_sym = mode == DG_MODE_VERTEX && algo == DG_WCC;
    const bool need_csr = mode == DG_MODE_VERTEX && !need_sym;
    const bool need_ew = (mode == DG_MODE_PATH && algo == DG_SSSP) || algo == DG_ADSORPTION;
    if ((need_sym || need_csr) && !g->layout.has_csr)
        return fail(DG_EINVAL, "dg_run: the vertex-centric ablation needs the CSR (this layout came from a file)");
    std::string err;
    try {
        if (need_sym) build_sym_csr(g->layout, g->csr.n);
    } catch (const std::bad_alloc&) {
        return fail(DG_ENOMEM, "dg_run: out of host memory (WCC ablation CSR)");
    }
    int rc = dg::dev_ensure_parts(g->dev, g->csr, g->layout, need_csr, need_ew, need_sym, err);
    return rc ? fail(rc, err) : DG_OK;
}



int dg_set_vertex_params(dg_graph* g, const double* p_inj, const double* p_cont, const double* inj) {
    if (!g || !g->layout.built) return fail(DG_EINVAL, "dg_set_vertex_params: no layout built");
    if (int rc0 = select_dev(g)) return rc0;
    if (int rc0 = ensure_uploaded(g)) return rc0;
    if (!p_inj || !p_cont || !inj) return fail(DG_EINVAL, "dg_set_vertex_params: NULL array");
    if (int rc0 = ensure_parts(g, DG_ADSORPTION, DG_MODE_PATH)) return rc0;
    for (int64_t v = 0; v < g->csr.n; v++)
        if (!(p_cont[v] >= 0 && p_cont[v] < 1 && p_inj[v] >= 0))
            return fail(DG_EINVAL, "dg_set_vertex_params: need 0 <= p_cont < 1 and p_inj >= 0");
    // to internal vertex ids
    const auto& orig = g->layout.orig;
    const int64_t n = g->csr.n;
    std::vector<double> a(n), b(n), c(n);
    for (int64_t u = 0; u < n; u++) { a[u] = p_inj[orig[u]]; b[u] = p_cont[orig[u]]; c[u] = inj[orig[u]]; }
    std::string err;
    int rc = dg::dev_set_vertex_params(g->work, g->dev, a.data(), b.data(), c.data(), g->layout.wsum.data(), err);
    return rc ? fail(rc, err) : DG_OK;
}

// SSSP/BFS bucket width from dg_run's param (include/digraph.h, reading R-DELTA)
static int64_t run_delta(const dg_graph* g, int algo, double param) {
    if (algo != DG_SSSP && algo != DG_BFS) return 0;
    if (param > 0) return (int64_t)param;
    if (param < 0) return 0;
    return algo == DG_SSSP ? 2 * (int64_t)g->csr.max_w : 1;  // BFS: level-synchronous
}

static int check_run_args(dg_graph* g, int algo, int64_t source, double epsilon, double param, int mode) {
    if (!g || !g->layout.built) return fail(DG_EINVAL, "dg_run: no layout built");
    if (algo < DG_SSSP || algo > DG_ADSORPTION) return fail(DG_EINVAL, "dg_run: unknown algorithm");
    if (mode != DG_MODE_PATH && mode != DG_MODE_VERTEX) return fail(DG_EINVAL, "dg_run: unknown mode");
    if ((algo == DG_SSSP || algo == DG_BFS) && (source < 0 || source >= g->csr.n))
        return fail(DG_EINVAL, "dg_run: source out of range");
    if (algo == DG_PAGERANK && !(param > 0 && param < 1)) return fail(DG_EINVAL, "dg_run: damping must be in (0,1)");
    if ((algo == DG_PAGERANK || algo == DG_ADSORPTION) && !(epsilon > 0))
        return fail(DG_EINVAL, "dg_run: epsilon must be > 0");
    if (mode == DG_MODE_VERTEX && algo != DG_SSSP && algo != DG_BFS && algo != DG_PAGERANK && algo != DG_WCC)
        return fail(DG_EINVAL, "dg_run: the vertex-centric ablation supports SSSP, BFS, PageRank and WCC");
    return DG_OK;
}

int dg_run(dg_graph* g, int algo, int64_t source, double epsilon, double param, int mode,
           int64_t max_rounds, dg_run_stats* stats) {
    int rc = check_run_args(g, algo, source, epsilon, param, mode);
    if (rc) return rc;
    if (g->layout.params.world > 1 && mode == DG_MODE_PATH)
        return fail(DG_EINVAL, "dg_run: multi-rank layout; use dg_run_begin/dg_rounds/dg_boundary_*");
    if ((rc = select_dev(g))) return rc;
    if ((rc = ensure_uploaded(g))) return rc;
    if ((rc = ensure_parts(g, algo, mode))) return rc;
    g->run = dg::RunState();
    g->run.algo = algo; g->run.mode = mode;
    g->run.source = (algo == DG_SSSP || algo == DG_BFS) ? g->layout.new_id[source] : 0;
    g->run.eps = epsilon; g->run.param = param;
    g->run.delta = run_delta(g, algo, param);
    std::string err;
    rc = dg::dev_run(g->work, g->dev, g->run, max_rounds <= 0 ? 1000000 : max_rounds, err);
    if (stats) *stats = g->run.stats;
    if (rc && rc != DG_ENOCONV) return fail(rc, err);
    g->ran = true;
    return rc ? fail(rc, err) : DG_OK;
}

int dg_get_states(dg_graph* g, void* out, int64_t n, int out_is_device) {
    if (!g || !g->ran) return fail(DG_EINVAL, "dg_get_states: nothing has run");
    if (int rc0 = select_dev(g)) return rc0;
    if (!out || n != g->csr.n) return fail(DG_EINVAL, "dg_get_states: out is NULL or n mismatch");
    std::string err;
    int rc = dg::dev_get_states(g->work, g->dev, g->run, out, n, out_is_device, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_normalize_states(dg_graph* g, void* buf, int64_t n) {
    if (!g || !buf || n < 0) return fail(DG_EINVAL, "dg_normalize_states: bad argument");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_normalize(buf, n, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_get_layout_info(const dg_graph* g, dg_layout_info* info) {
    if (!g || !info) return fail(DG_EINVAL, "dg_get_layout_info: NULL argument");
    std::memset(info, 0, sizeof(*info));
    info->n = g->csr.n;
    info->m = g->csr.m;
    const auto& L = g->layout;
    if (!L.built) return DG_OK;
    info->n_paths = (int64_t)L.path_off.size() - 1;
    info->n_entries = (int64_t)L.e_idx.size();
    info->n_partitions = (int64_t)L.part_off.size() - 1;
    info->n_hot_paths = L.n_hot;
    info->n_layers = L.n_layers;
    info->n_dep_sccs = L.n_dep_sccs;
    info->giant_scc_paths = L.giant;
    info->n_boundary = (int64_t)L.boundary.size();
    info->paths_before_merge = L.paths_before_merge;
    info->preprocess_ms = L.preprocess_ms;
    info->device_bytes = g->dev.bytes;
    info->h2d_bytes = g->dev.h2d_bytes;
    const int rk = L.params.rank;
    for (const uint64_t h : L.bnd_hold)
        if ((h >> rk) & 1ull) info->boundary_reads += __builtin_popcountll(h) - 1;
    if (L.hub_entries < 0) {
        const uint32_t H = (uint32_t)std::max<int64_t>(0, L.n_proxy);
        const int64_t M = (int64_t)L.e_idx.size();
        int64_t c = 0;
#pragma omp parallel for reduction(+ : c) schedule(static)
        for (int64_t k = 0; k < M; k++) c += (L.e_idx[k] & dg::kVMask) < H;
        L.hub_entries = c;
    }
    info->hub_entries = L.hub_entries;
    return DG_OK;
}

int dg_export_paths(const dg_graph* g, int64_t* path_off, int32_t* vertices, int32_t* layer, int64_t* scc,
                    int64_t* merged_index, uint8_t* hot, int64_t* part_off) {
    if (!g || !g->layout.built) return fail(DG_EINVAL, "dg_export_paths: no layout built");
    const auto& L = g->layout;
    const size_t P = L.path_off.size() - 1;
    if (path_off) std::memcpy(path_off, L.path_off.data(), sizeof(int64_t) * (P + 1));
    if (vertices)
        for (size_t k = 0; k < L.e_idx.size(); k++) vertices[k] = L.orig[L.e_idx[k] & dg::kVMask];
    if (layer) std::memcpy(layer, L.layer.data(), sizeof(int32_t) * P);
    if (scc) std::memcpy(scc, L.scc.data(), sizeof(int64_t) * P);
    if (merged_index) std::memcpy(merged_index, L.merged_index.data(), sizeof(int64_t) * P);
    if (hot) std::memcpy(hot, L.hot.data(), P);
    if (part_off) std::memcpy(part_off, L.part_off.data(), sizeof(int64_t) * L.part_off.size());
    return DG_OK;
}

int dg_boundary_size(const dg_graph* g, int64_t* n_boundary) {
    if (!g || !g->layout.built || !n_boundary) return fail(DG_EINVAL, "dg_boundary_size: no layout built");
    *n_boundary = (int64_t)g->layout.boundary.size();
    return DG_OK;
}

int dg_boundary_vertices(const dg_graph* g, int32_t* out) {
    if (!g || !g->layout.built || !out) return fail(DG_EINVAL, "dg_boundary_vertices: no layout built");
    std::vector<int32_t> b(g->layout.boundary.size());
    for (size_t k = 0; k < b.size(); k++) b[k] = g->layout.orig[g->layout.boundary[k]];
    std::sort(b.begin(), b.end());
    std::memcpy(out, b.data(), sizeof(int32_t) * b.size());
    return DG_OK;
}

int dg_run_begin(dg_graph* g, int algo, int64_t source, double epsilon, double param) {
    int rc = check_run_args(g, algo, source, epsilon, param, DG_MODE_PATH);
    if (rc) return rc;
    if ((rc = select_dev(g))) return rc;
    if ((rc = ensure_uploaded(g))) return rc;
    if ((rc = ensure_parts(g, algo, DG_MODE_PATH))) return rc;
    g->run = dg::RunState();
    g->run.algo = algo; g->run.mode = DG_MODE_PATH;
    g->run.source = (algo == DG_SSSP || algo == DG_BFS) ? g->layout.new_id[source] : 0;
    g->run.eps = epsilon; g->run.param = param;
    g->run.delta = run_delta(g, algo, param);
    g->run.raw_states = g->layout.params.world > 1;
    std::string err;
    rc = dg::dev_run_begin(g->work, g->dev, g->run, err);
    if (rc) return fail(rc, err);
    g->multi_active = true;
    return DG_OK;
}

int dg_scc_phase(dg_graph* g, int phase, int64_t* active) {
    if (!g || !g->multi_active || g->run.algo != DG_SCC || !active || (phase != 0 && phase != 1))
        return fail(DG_EINVAL, "dg_scc_phase: no multi-rank SCC run in progress, or phase not 0/1");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_scc_phase(g->work, g->dev, g->run, phase, active, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_scc_assign(dg_graph* g, int64_t* remaining) {
    if (!g || !g->multi_active || g->run.algo != DG_SCC || !remaining)
        return fail(DG_EINVAL, "dg_scc_assign: no multi-rank SCC run in progress");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_scc_assign(g->work, g->dev, g->run, remaining, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_rounds(dg_graph* g, int64_t max_rounds, int64_t* active) {
    if (!g || !g->multi_active || !active) return fail(DG_EINVAL, "dg_rounds: no run in progress");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_rounds(g->work, g->dev, g->run, max_rounds <= 0 ? 1000000 : max_rounds, active, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_boundary_pack(dg_graph* g, void* buf) {
    if (!g || !g->multi_active) return fail(DG_EINVAL, "dg_boundary_pack: no run in progress");
    if (int rc0 = select_dev(g)) return rc0;
    if (!buf && !g->layout.boundary.empty()) return fail(DG_EINVAL, "dg_boundary_pack: NULL buffer");
    std::string err;
    int rc = dg::dev_boundary_pack(g->work, g->dev, g->run, buf, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_boundary_unpack(dg_graph* g, const void* buf, int64_t* active) {
    if (!g || !g->multi_active || !active) return fail(DG_EINVAL, "dg_boundary_unpack: no run in progress");
    if (int rc0 = select_dev(g)) return rc0;
    if (!buf && !g->layout.boundary.empty()) return fail(DG_EINVAL, "dg_boundary_unpack: NULL buffer");
    std::string err;
    int rc = dg::dev_boundary_unpack(g->work, g->dev, g->run, buf, active, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_p2p_alloc(dg_graph* g, int world, int rank, void* handle) {
    if (!g || !g->layout.built || !handle) return fail(DG_EINVAL, "dg_p2p_alloc: no layout built or NULL handle");
    if (!g->uploaded) return fail(DG_EINVAL, "dg_p2p_alloc: dg_upload first");
    if (world != g->layout.params.world || rank != g->layout.params.rank)
        return fail(DG_EINVAL, "dg_p2p_alloc: world/rank differ from the layout's (dg_build_paths)");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_p2p_alloc(g->p2p, g->dev, world, rank, handle, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_p2p_open(dg_graph* g, const void* handles) {
    if (!g || !handles) return fail(DG_EINVAL, "dg_p2p_open: NULL argument");
    if (!g->p2p) return fail(DG_EINVAL, "dg_p2p_open: dg_p2p_alloc first");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_p2p_open(g->p2p, handles, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_boundary_exchange(dg_graph* g, int64_t* active) {
    if (!g || !g->multi_active || !active) return fail(DG_EINVAL, "dg_boundary_exchange: no run in progress");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_boundary_exchange(g->work, g->dev, g->run, g->p2p, active, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_run_fused(dg_graph* g, int64_t local_rounds, int64_t max_rounds, int64_t* exchanges, int64_t* converged) {
    if (!g || !g->multi_active || !exchanges || !converged) return fail(DG_EINVAL, "dg_run_fused: no run in progress");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_run_fused(g->work, g->dev, g->run, g->p2p, local_rounds, max_rounds <= 0 ? 1000000 : max_rounds,
                               exchanges, converged, err);
    return rc ? fail(rc, err) : DG_OK;
}

int dg_run_end(dg_graph* g, dg_run_stats* stats) {
    if (!g || !g->multi_active) return fail(DG_EINVAL, "dg_run_end: no run in progress");
    if (int rc0 = select_dev(g)) return rc0;
    std::string err;
    int rc = dg::dev_run_end(g->work, g->dev, g->run, err);
    g->multi_active = false;
    if (rc) return fail(rc, err);
    g->ran = true;
    if (stats) *stats = g->run.stats;
    return DG_OK;
}

}  // extern "C"

static int select_dev(dg_graph* g) {
    std::string err;
    int rc = dg::dev_select(g->device, err);
    return rc ? fail(rc, err) : DG_OK;
}
