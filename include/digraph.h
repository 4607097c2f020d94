/*
 * digraph.h -- C ABI of the B200-native DiGraph hot path.
 *
 * DiGraph (Zhang et al., ASPLOS'19; /root/reference/PAPER.md) processes an
 * iterative directed-graph algorithm by splitting the graph into disjoint
 * directed paths and propagating vertex states along each path inside one
 * round ("path-based asynchronous execution", sec. 3.1, lines
 * 88-102).  This header is the boundary between the (thin) Python binding and
 * the native library libdigraph.so: plain C types, plain pointers and sizes.
 *
 * Conventions (all functions):
 *   - return 0 on success, a negative DG_E* code on failure; the message of
 *     the last failure on the calling thread is dg_last_error();
 *   - no function falls back to the CPU for a computation step: when the
 *     CUDA device or the kernels are unavailable the call fails with
 *     DG_ENOCUDA;
 *   - pointers documented as HOST are ordinary host memory (pageable or
 *     pinned) and are only read/written during the call; DEVICE pointers
 *     are CUDA device pointers on the graph's device;
 *   - the library never takes ownership of caller memory.
 *
 * Lifecycle: dg_create -> dg_load_csr -> dg_build_paths -> (dg_run ->
 * dg_get_states)* -> dg_destroy.
 */
#ifndef DIGRAPH_H
#define DIGRAPH_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define DG_OK 0
#define DG_EINVAL (-1)   /* bad argument / wrong lifecycle order            */
#define DG_ENOMEM (-2)   /* host or device allocation failed                */
#define DG_ENOCUDA (-3)  /* no CUDA device / kernel launch failed           */
#define DG_ENOCONV (-4)  /* max_rounds reached before convergence           */
#define DG_ETIMEOUT (-5) /* a peer rank never reached a boundary exchange  */

/* Unreachable vertex distance for SSSP/BFS (reading R-INF). */
#define DG_INF 0x7FFFFFFFu

/* Algorithms (sec. 4 benchmarks + BASELINE.json north_star). */
typedef enum {
    DG_SSSP = 0,       /* min-plus relaxation, integer weights >= 0           */
    DG_BFS = 1,        /* SSSP with unit weights                              */
    DG_PAGERANK = 2,   /* delta-accumulative PageRank, d = `param`           */
    DG_WCC = 3,        /* min-label propagation over both edge directions     */
    DG_SCC = 4,        /* forward colouring + backward reachability rounds    */
    DG_ADSORPTION = 5  /* accumulative Adsorption (dg_set_vertex_params)      */
} dg_algo;

/* Execution model. */
typedef enum {
    DG_MODE_PATH = 0,    /* DiGraph path-based asynchronous model (the product) */
    DG_MODE_VERTEX = 1   /* vertex-centric frontier kernel (ablation baseline)  */
} dg_mode;

typedef struct dg_graph dg_graph;

/* Parameters of the preprocessing rows (sec. 3.2.1, 3.2.3). */
typedef struct {
    int32_t d_max;         /* DFS depth bound D_MAX of Algorithm 1 (line 3); paper default 16 */
    int32_t l_merge;       /* max edges of a merged path (reading R-MERGE); 0 = no merge */
    int32_t n_sub;         /* number of subgraphs Algorithm 1 runs on in parallel (line 114) */
    int32_t order;         /* successor/root order: 0 = degree desc (line 5), 1 = vertex id */
    float hot_factor;      /* hot path iff avg degree >= hot_factor * mean degree (R-HOT) */
    int32_t part_entries;  /* target path entries per partition (scheduling unit); 0 = auto
                              (about 16K partitions, 512..2048 entries each) */
    int32_t rank;          /* this process's rank for multi-GPU path partitioning */
    int32_t world;         /* number of ranks (1 = single GPU) */
    int32_t merge_rule;    /* 0: paper-literal (no merge through a line-13 inner vertex of
                              in/out degree > 1); 1: relaxed (any head-to-tail merge within
                              l_merge; reading R-MERGE) */
    int32_t n_proxy;       /* highest-degree vertices kept as shared-memory proxies by the
                              PageRank/Adsorption walk; 0 = none */
    int32_t placement;     /* world > 1: partition -> rank placement; 0: round-robin over the
                              priority order; 1: locality (each partition to the rank already
                              holding most of its vertices, entry loads within 2 %; PAPER.md
                              line 178; reading R-PLACE) */
} dg_path_params;

/* Fill *p with the defaults (d_max 16, l_merge 64, n_sub 64, order 0,
 * hot_factor 2, part_entries 0 (auto), rank 0, world 1, merge_rule 1,
 * n_proxy 8192 (the kernel uses as many as fit its shared memory),
 * placement 1). */
void dg_default_params(dg_path_params *p);

/* Statistics of one dg_run (device-side counters). */
typedef struct {
    double time_ms;               /* device time of the run (CUDA events)          */
    int64_t rounds;               /* rounds until the active counter reached zero  */
    int64_t vertex_updates;       /* master-state changes (successful relax/fold)  */
    int64_t edges_processed;      /* path edges (or CSR edges) walked              */
    int64_t units_processed;      /* 128-entry windows walked (path) / vertices expanded (vertex) */
    int64_t kernel_launches;      /* kernels launched by this run                  */
    int64_t outer_iterations;     /* SCC colouring iterations (0 otherwise)        */
    int64_t entries_processed;    /* path entries walked (path mode)               */
    int64_t csr_edges;            /* CSR out-edges pushed (delta algorithms, ablation) */
    double kernel_ms;             /* device time of the propagation kernels only   */
    int64_t dense_rounds;         /* path mode: rounds that streamed every window's
                                     entries (the others walked sparse from the
                                     signalled vertices); for the byte model      */
} dg_run_stats;

/* Static description of the built layout (sizes; for tests and benchmarks). */
typedef struct {
    int64_t n, m;                 /* vertices, edges                                */
    int64_t n_paths;              /* paths after merging (this rank)                */
    int64_t n_entries;            /* path entries = sum(len+1) (this rank)          */
    int64_t n_partitions;         /* partitions (this rank)                         */
    int64_t n_hot_paths;          /* hot paths (this rank)                          */
    int64_t n_layers;             /* layers of the DAG sketch                       */
    int64_t n_dep_sccs;           /* SCCs of the path dependency graph containing paths */
    int64_t giant_scc_paths;      /* paths in the largest dependency SCC            */
    int64_t n_boundary;           /* vertices replicated on >1 rank                 */
    int64_t paths_before_merge;   /* paths produced by Algorithm 1                  */
    double preprocess_ms;         /* host time of dg_build_paths                    */
    int64_t device_bytes;         /* device memory held by the layout               */
    int64_t h2d_bytes;            /* bytes the last dg_upload copied host -> device */
    int64_t boundary_reads;       /* peer slots this rank reads per peer-memory exchange:
                                     sum over the boundary vertices its paths hold of
                                     (ranks holding the vertex - 1); x 8 B = NVLink bytes */
    int64_t hub_entries;          /* path entries of the n_proxy highest-degree vertices
                                     (the shared-memory proxies of PageRank/Adsorption) */
} dg_layout_info;

/* Create an empty graph bound to CUDA device `device` (cudaSetDevice is
 * called on entry of every function).  *out receives the handle. */
int dg_create(dg_graph **out, int device);

/* Destroy a graph and free all host and device memory it holds. */
void dg_destroy(dg_graph *g);

/* Thread-local message of the last failure ("" if none). */
const char *dg_last_error(void);

/* Load a directed graph in CSR form (sec. 3.1: G = (V, E)).
 *   n        number of vertices (ids 0..n-1, n < 2^30)
 *   m        number of directed edges
 *   row_ptr  HOST int64[n+1], non-decreasing, row_ptr[0] = 0, row_ptr[n] = m
 *   col      HOST int32[m], destination of edge k (source = the row)
 *   weight   HOST int32[m] edge weights (>= 0) or NULL (all weights 1)
 * The arrays are copied (host copy for preprocessing, device copy for the
 * vertex-centric ablation).  On success it invalidates a previous graph,
 * layout and device state; on failure (DG_EINVAL / DG_ENOMEM) the handle is
 * left exactly as it was. */
int dg_load_csr(dg_graph *g, int64_t n, int64_t m, const int64_t *row_ptr,
                const int32_t *col, const int32_t *weight);

/* Build the path layout on the host (C++, OpenMP; no device needed):
 * Algorithm 1 path decomposition, short-path
 * merging (line 157), hot/cold classification (line 112), path dependency
 * graph + Tarjan SCC condensation + layering (lines 98-102, 159, 169),
 * priority order Pri(p) (line 192), partitions (line 161/163) and, when
 * p->world > 1, the partitions owned by p->rank plus the boundary-vertex set
 * ("state synchronization of vertex replicas").
 * p may be NULL (defaults). */
int dg_build_paths(dg_graph *g, const dg_path_params *p);

/* ---- preprocess once, hand every rank its share (PAPER.md lines 104-114,
 * 176: the graph is preprocessed on the CPU, then paths are dispatched from
 * the host to the GPUs) ----
 * dg_build_paths_shared: ONE preprocessing pass for all p->world ranks; writes
 *   rank r's layout to the file "<prefix>.<r>" (r = 0..world-1) and keeps
 *   rank p->rank's layout in this handle (as dg_build_paths would).  The
 *   caller owns the files (e.g. under /dev/shm) and removes them.
 * dg_save_layout: write this handle's built layout to `path`.
 * dg_load_layout: replace this handle's graph and layout with a layout file
 *   (then dg_upload / dg_run as usual; no dg_load_csr is needed).  A loaded
 *   layout carries no CSR: dg_build_paths and the vertex-centric ablation
 *   return DG_EINVAL on it; every path-mode algorithm runs.  On failure the
 *   handle is unchanged.
 * Files are host byte order with a version tag (DG_EINVAL on mismatch,
 * truncation or an unopenable path). */
int dg_build_paths_shared(dg_graph *g, const dg_path_params *p, const char *prefix);
int dg_save_layout(const dg_graph *g, const char *path);
int dg_load_layout(dg_graph *g, const char *path);

/* Copy the host CSR and the built layout to the device (the H2D part of an
 * end-to-end run).  dg_run / dg_run_begin / dg_set_vertex_params call it
 * implicitly when the layout is not on the device yet.  Fails with
 * DG_ENOCUDA when no CUDA device is present. */
int dg_upload(dg_graph *g);

/* Per-vertex inputs of Adsorption (reading R-ADS):
 *   p_inj, p_cont, inj  HOST double[n]; x_v = p_inj*inj + sum p_cont(u) w(u,v)/W(u) x_u.
 * Must be called before dg_run(DG_ADSORPTION). */
int dg_set_vertex_params(dg_graph *g, const double *p_inj, const double *p_cont,
                         const double *inj);

/* Run `algo` to convergence on the device.
 *   source   SSSP/BFS source vertex (ignored otherwise)
 *   epsilon  PageRank/Adsorption per-vertex stop threshold on the delta
 *            (north_star: 1e-7 with unnormalised ranks (1-d) + d*sum);
 *            ignored by the exact algorithms
 *   param    PageRank: damping d (0 < d < 1).
 *            SSSP/BFS: bucket width Delta of the rounds (DESIGN.md reading
 *            R-DELTA): a round commits only distances <= (smallest distance
 *            signalled by the previous round) + Delta.  0 = library default
 *            (SSSP: 2 * max edge weight; BFS: 1, level-synchronous),
 *            < 0 = unbounded,
 *            > 0 = that width (values above 2^31-1 act as unbounded).
 *            Results are exact for every value; it trades redundant
 *            updates against rounds.  Ignored by the others.
 *   mode     DG_MODE_PATH or DG_MODE_VERTEX (ablation: SSSP, BFS, PageRank,
 *            WCC -- WCC pushes labels over both edge directions)
 *   max_rounds  safety cap (<= 0: 1,000,000)
 *   stats    may be NULL
 * DG_ENOCONV if max_rounds ended the run (for SCC: any forward or backward
 * phase) before convergence; the states are then not final.
 * States stay on the device until dg_get_states.  Single-rank only: with
 * world > 1 use dg_rounds / dg_boundary_* (multi-GPU protocol). */
int dg_run(dg_graph *g, int algo, int64_t source, double epsilon, double param,
           int mode, int64_t max_rounds, dg_run_stats *stats);

/* Copy the final states of the last dg_run into `out` (n elements):
 *   SSSP/BFS      uint32 distances (DG_INF unreachable)
 *   PAGERANK      float32 ranks normalised to sum 1 (reading R-PR);
 *                 after a multi-rank run (world > 1): this rank's unnormalised
 *                 totals -- take the MAX over ranks (totals grow monotonically
 *                 from the same initial value), then dg_normalize_states
 *   ADSORPTION    float32 scores x_v
 *   WCC / SCC     int32 label = smallest vertex id of the component
 *   out_is_device 0: `out` is HOST memory; 1: DEVICE memory. */
int dg_get_states(dg_graph *g, void *out, int64_t n, int out_is_device);

/* Normalise a DEVICE float32[n] buffer in place to sum 1 (the last step of a
 * multi-rank PageRank after the contributions were summed over ranks). */
int dg_normalize_states(dg_graph *g, void *buf, int64_t n);

/* Layout sizes / preprocessing time. */
int dg_get_layout_info(const dg_graph *g, dg_layout_info *info);

/* Export the built paths (this rank, priority order) for validation:
 *   path_off  HOST int64[n_paths+1] (may be NULL to query only)
 *   vertices  HOST int32[n_entries]: vertices of each path in path order
 *   layer     HOST int32[n_paths] layer number L(p) (may be NULL)
 *   scc       HOST int64[n_paths] canonical SCC label: smallest merged-order
 *             index of a path in the same dependency SCC (may be NULL)
 *   merged_index HOST int64[n_paths] index of the path in merge order (may be NULL)
 *   hot       HOST uint8[n_paths] hot flag (may be NULL)
 *   part_off  HOST int64[n_partitions+1] partition -> entry offsets (may be NULL) */
int dg_export_paths(const dg_graph *g, int64_t *path_off, int32_t *vertices, int32_t *layer,
                    int64_t *scc, int64_t *merged_index, uint8_t *hot, int64_t *part_off);

/* ---- multi-GPU protocol (one process per GPU; PyTorch/NCCL moves bytes) ----
 * A run is: dg_round_begin, then repeat { dg_rounds (local rounds until the
 * local active counter is zero or max_rounds); dg_boundary_pack;
 * all-reduce the buffer across ranks (MIN for SSSP/BFS/WCC, SUM for
 * PageRank/Adsorption); dg_boundary_unpack } until the all-reduced active
 * count is zero; dg_run_end. */

/* Number of boundary vertices (vertices on more than one rank's paths).
 * Buffer elements: uint32 (as int32) for MIN algorithms, uint64 fixed-point
 * (2^-32 units, as int64) for SUM algorithms. */
int dg_boundary_size(const dg_graph *g, int64_t *n_boundary);

/* Export the boundary vertex ids (HOST int32[n_boundary], ascending). */
int dg_boundary_vertices(const dg_graph *g, int32_t *out);

/* Start a multi-round run (resets states as dg_run does). */
int dg_run_begin(dg_graph *g, int algo, int64_t source, double epsilon, double param);

/* Run up to max_rounds local rounds; *active is non-zero iff work remains
 * (an upper bound on the vertices signalled for the next round: a vertex
 * lowered twice in a round may count twice). */
int dg_rounds(dg_graph *g, int64_t max_rounds, int64_t *active);

/* Pack boundary states into DEVICE buffer `buf` (n_boundary elements, see
 * dg_boundary_size): MIN algorithms: the current states; SUM algorithms: the
 * growth of each total since the last unpack ("each mirror
 * always sends its new state to its master"). */
int dg_boundary_pack(dg_graph *g, void *buf);

/* Apply the all-reduced DEVICE buffer; vertices whose state changed are
 * signalled for the next local round.  *active is non-zero iff work remains
 * (an upper bound on the signalled vertices, as for dg_rounds). */
int dg_boundary_unpack(dg_graph *g, const void *buf, int64_t *active);

/* Multi-rank SCC (DG_SCC in dg_run_begin; the paths of an
 * SCC-vertex run "over SMXs of multiple GPUs"): the colouring iterations of
 * the single-rank dg_run(DG_SCC) with every phase a multi-rank run.  The
 * caller repeats { dg_scc_phase(0): forward min-colour propagation -- then
 * rounds and exchanges as for MIN algorithms (dg_rounds + dg_boundary_*,
 * dg_boundary_exchange or dg_run_fused) until the global activity is 0;
 * dg_scc_phase(1): the roots (vertices keeping their own id) start backward
 * reachability inside their colour -- rounds and exchanges again (the
 * replicated state is now the mark, packed as 0 = marked / 1 = not, so the
 * MIN exchange is an OR); dg_scc_assign: marked vertices take their colour
 * as label, *remaining = this rank's unassigned vertices } until the sum of
 * `remaining` over ranks is 0; then dg_run_end.  *active = vertices the phase
 * signalled on this rank.  dg_get_states then returns this rank's labels; a
 * vertex on none of its paths carries its own id, so the MIN over ranks is
 * every vertex's label (smallest vertex id of its SCC). */
int dg_scc_phase(dg_graph *g, int phase, int64_t *active);
int dg_scc_assign(dg_graph *g, int64_t *remaining);

/* Finish the run: normalisation (PageRank) and statistics. */
int dg_run_end(dg_graph *g, dg_run_stats *stats);

/* ---- peer-memory boundary exchange (replaces pack + all-reduce + unpack) ----
 * PAPER.md line 96 ("state propagation between paths is done through state
 * synchronization of vertex replicas ... in batches") and line 184 (mirrors
 * send their new states to their masters).  Every rank owns one exchange
 * region in its own device memory (256 B of epoch flags + 2 x n_boundary
 * uint64 slots), mapped into every other rank by CUDA IPC; an exchange packs
 * this rank's boundary values into its slot, publishes an epoch number into
 * every peer's flag word, waits (on the device) for every peer's epoch, then
 * reduces all ranks' slots elementwise straight from peer memory (MIN for
 * SSSP/BFS/WCC, SUM of fixed-point growth for PageRank/Adsorption) and
 * applies the result like dg_boundary_unpack.  No host collective moves the
 * boundary states.  All ranks must hold the same layout (same boundary set)
 * and call dg_boundary_exchange the same number of times.
 *
 * dg_p2p_alloc: after dg_build_paths(rank, world) and dg_upload; allocates
 *   the region (the library owns it; freed by dg_destroy or the next
 *   dg_p2p_alloc) and writes its IPC handle to HOST `handle` (64 bytes).
 *   2 <= world <= 16; world and rank must be the layout's (dg_build_paths).
 *   The caller distributes the handles (any transport).
 * dg_p2p_open: HOST `handles` = world x 64 bytes in rank order (this rank's
 *   own entry is ignored); maps every peer's region.  Ranks on the same GPU
 *   in different processes are allowed (tests); two ranks in one process are
 *   not (CUDA IPC).
 * dg_boundary_exchange: during a run (after dg_rounds); *active = vertices
 *   this rank re-signalled.  DG_ETIMEOUT if a peer has not arrived after 60 s
 *   (the device wait gives up instead of hanging). */
int dg_p2p_alloc(dg_graph *g, int world, int rank, void *handle);
int dg_p2p_open(dg_graph *g, const void *handles);
int dg_boundary_exchange(dg_graph *g, int64_t *active);

/* The whole multi-rank run in ONE kernel launch per rank (after
 * dg_run_begin and dg_p2p_open, before dg_run_end): the persistent
 * propagation kernel performs the same peer-memory exchange itself after
 * every `local_rounds` rounds (or as soon as this rank has no work), and
 * stops when every rank published zero activity (no signalled vertex and
 * no boundary value changed since the previous exchange) at the same
 * exchange -- the global convergence test runs on the devices, no host
 * collective.  SSSP, BFS, WCC, PageRank, Adsorption.  Every rank must call
 * it together (the kernels rendezvous through the epoch flags).
 *   *exchanges  exchanges performed; *converged 1 if globally converged
 *   (0: max_rounds reached).  DG_ETIMEOUT if a peer did not arrive within
 *   60 s. */
int dg_run_fused(dg_graph *g, int64_t local_rounds, int64_t max_rounds, int64_t *exchanges, int64_t *converged);

#ifdef __cplusplus
}
#endif
#endif /* DIGRAPH_H */
