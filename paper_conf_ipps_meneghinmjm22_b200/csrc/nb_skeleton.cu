// nb_skeleton.cu — the Skeleton: sequential user code (a list of map /
// stencil / reduce Containers) -> data-dependency graph -> multi-GPU graph
// with halo nodes and OCC splits -> stream / event / task-order schedule ->
// execution (§V).
//
// Planning is pure host C++ (nb_skeleton_plan is callable without a GPU);
// execution enqueues the library's own kernels (axpby, laplace7, the
// canonical dot) on the planned streams.  The hand-written fused schedules
// (nb_map_stencil_reduce, the CG) are the ground truth: a generated schedule
// must give the same bits (tests/test_gpu_skeleton.py).
//
// Steps, in the paper's order:
//  A. Data dependency graph (L279-L290).  Nodes = Containers with an
//     operation type (MapOp / StencilOp / ReduceOp), a data view and a
//     coherency flag (a stencil whose input halo is stale).  Edges join
//     nodes that touch the same data with at least one write (RaW, WaR,
//     WaW).  Data is tracked per field and per plane class of a slab
//     (halo below, boundary plane below, core, boundary plane above, halo
//     above), so split nodes get exact dependencies.
//  B. Multi-GPU graph (L292-L331): a halo-update node before every
//     incoherent stencil; OCC splits — STANDARD splits the stencil into
//     Internal / Boundary, EXTENDED also splits the maps feeding it,
//     TWO_WAY also the maps / reduces consuming it (reduce Internal ->
//     reduce Boundary dependency added); redundant (transitively implied)
//     edges removed; scheduling hints "launch the internal nodes before the
//     halo node" (L318-L330).
//  C. Scheduling (L333-L396): BFS levels over the data edges, one stream
//     per concurrent node of the widest level, a node reuses a parent's
//     stream when it can; an event for every cross-stream data edge; task
//     order = BFS levels over data edges + hints.
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <functional>
#include <queue>
#include <string>
#include <vector>

#include "nb_internal.cuh"

nb_status nb_dot_partials_view(const nb_field *x, const nb_field *y, nb_view v);
std::vector<std::pair<int, int>> view_ranges(const nb_grid *g, int p, nb_view v);

namespace {

// plane classes of a slab (radius 1)
enum : int { R_HLO = 1, R_BLO = 2, R_CORE = 4, R_BHI = 8, R_HHI = 16 };
constexpr int R_OWN = R_BLO | R_CORE | R_BHI, R_ALL = R_OWN | R_HLO | R_HHI;

enum SkOp { SK_MAP = 0, SK_STENCIL = 1, SK_REDUCE = 2, SK_HALO = 3, SK_SCALAR = 4 };
const char *op_name(int op) {
    static const char *n[] = {"map", "stencil", "reduce", "halo", "scalar"};
    return n[op];
}
// StencilOps read their input's halo (radius 1)
bool is_stencil(int op) { return op == NB_SK_LAPLACE7 || op == NB_SK_POISSON || op == NB_SK_LBM; }
const char *view_name(nb_view v) {
    static const char *n[] = {"standard", "internal", "boundary"};
    return n[v];
}

int view_mask(nb_view v) { return v == NB_VIEW_STANDARD ? R_OWN : (v == NB_VIEW_INTERNAL ? R_CORE : R_BLO | R_BHI); }
// planes a radius-1 stencil over view v reads
int stencil_read_mask(nb_view v) {
    return v == NB_VIEW_STANDARD ? R_ALL : (v == NB_VIEW_INTERNAL ? R_OWN : R_ALL);
}

struct Access {
    int field;  // field id, or SCALAR_BASE + slot, or TP_FIELD (reduction scratch)
    int mask;
    bool write;
};

constexpr int TP_FIELD = 1 << 20;      // the grid's shared reduction scratch
constexpr int SCALAR_BASE = 1 << 21;   // dot result slots

struct Node {
    int id = 0;
    int op = SK_MAP;
    nb_view view = NB_VIEW_STANDARD;
    int container = -1;   // index of the user Container (-1: halo node)
    int halo_field = -1;  // halo nodes
    bool halo_lbm = false;  // halo of an LBM container: the 5 + 5 z-crossing populations
    bool incoherent = false;
    bool finalize = false;  // reduce part that completes the reduction
    std::vector<Access> acc;
    int level = 0, stream = 0, event = -1;
    std::vector<int> waits;
    std::string name;
};

struct Plan {
    std::vector<Node> nodes;
    std::vector<std::pair<int, int>> data, hints;
    std::vector<int> order;
    int nstreams = 0, nevents = 0;
};

bool conflict(const Node &a, const Node &b) {
    for (const Access &x : a.acc)
        for (const Access &y : b.acc)
            if (x.field == y.field && (x.mask & y.mask) && (x.write || y.write)) return true;
    return false;
}

// reachability over the given adjacency (DFS)
bool reaches(const std::vector<std::vector<int>> &adj, int from, int to, int skip_edge_to = -1) {
    std::vector<char> seen(adj.size(), 0);
    std::vector<int> st{from};
    while (!st.empty()) {
        int u = st.back();
        st.pop_back();
        for (int v : adj[u]) {
            if (u == from && v == skip_edge_to) continue;
            if (v == to) return true;
            if (!seen[v]) {
                seen[v] = 1;
                st.push_back(v);
            }
        }
    }
    return false;
}

// Kahn BFS levels; returns false on a cycle
bool bfs_levels(int n, const std::vector<std::pair<int, int>> &edges, std::vector<int> &level,
                std::vector<std::vector<int>> &levels) {
    std::vector<std::vector<int>> out(n);
    std::vector<int> indeg(n, 0);
    for (auto &e : edges) {
        out[e.first].push_back(e.second);
        indeg[e.second]++;
    }
    level.assign(n, 0);
    levels.clear();
    std::vector<int> frontier;
    for (int i = 0; i < n; ++i)
        if (!indeg[i]) frontier.push_back(i);
    int done = 0;
    while (!frontier.empty()) {
        std::sort(frontier.begin(), frontier.end());
        levels.push_back(frontier);
        std::vector<int> next;
        for (int u : frontier) {
            level[u] = (int)levels.size() - 1;
            ++done;
            for (int v : out[u])
                if (--indeg[v] == 0) next.push_back(v);
        }
        frontier.swap(next);
    }
    return done == n;
}

// A. + B.: nodes with accesses, halo nodes, OCC splits
nb_status build_nodes(const nb_container *c, int n, int nparts, nb_occ occ, Plan &P) {
    const bool multi = nparts > 1;  // a single slab has no inter-partition halo
    // which containers get split (Internal + Boundary)
    std::vector<char> split(n, 0), incoh(n, 0);
    std::vector<int> halo_before(n, -1);  // field whose halo precedes container i
    // coherency: a field's halo is current after a halo node until written
    std::vector<int> coherent_fields;  // fields with current halos
    auto is_coh = [&](int f) { return std::find(coherent_fields.begin(), coherent_fields.end(), f) != coherent_fields.end(); };
    auto set_coh = [&](int f, bool on) {
        auto it = std::find(coherent_fields.begin(), coherent_fields.end(), f);
        if (on && it == coherent_fields.end()) coherent_fields.push_back(f);
        if (!on && it != coherent_fields.end()) coherent_fields.erase(it);
    };
    for (int i = 0; i < n; ++i) {
        if (c[i].op < NB_SK_AXPBY || c[i].op > NB_SK_LBM) NB_FAIL(NB_EINVAL, "container %d: bad op %d", i, c[i].op);
        if (c[i].op == NB_SK_SCALAR) {
            if (c[i].sop < NB_SC_DIV || c[i].sop > NB_SC_SET) NB_FAIL(NB_EINVAL, "container %d: bad scalar op", i);
            if (c[i].slot < 0 || c[i].slot >= NB_DOT_SLOTS || c[i].x < 0 || c[i].x >= NB_DOT_SLOTS || c[i].y < 0 ||
                c[i].y >= NB_DOT_SLOTS)
                NB_FAIL(NB_EINVAL, "container %d: scalar slot out of range", i);
            continue;
        }
        if (c[i].x < 0 || c[i].y < 0 || c[i].x >= TP_FIELD || c[i].y >= TP_FIELD)
            NB_FAIL(NB_EINVAL, "container %d: bad field ids", i);
        if (is_stencil(c[i].op) && c[i].x == c[i].y) NB_FAIL(NB_EINVAL, "container %d: stencil in place", i);
        if (c[i].op == NB_SK_DOT && (c[i].slot < 0 || c[i].slot >= NB_DOT_SLOTS))
            NB_FAIL(NB_EINVAL, "container %d: slot out of range", i);
        if (c[i].op == NB_SK_AXPBY && (c[i].a_slot >= NB_DOT_SLOTS || c[i].b_slot >= NB_DOT_SLOTS))
            NB_FAIL(NB_EINVAL, "container %d: coefficient slot out of range", i);
        if (is_stencil(c[i].op)) {
            if (multi && !is_coh(c[i].x)) {
                incoh[i] = 1;
                halo_before[i] = c[i].x;
                set_coh(c[i].x, true);
            }
            set_coh(c[i].y, false);
        } else if (c[i].op == NB_SK_AXPBY) {
            set_coh(c[i].y, false);
        }
    }
    if (multi && occ != NB_OCC_NONE) {
        for (int i = 0; i < n; ++i) {
            if (!incoh[i]) continue;
            split[i] = 1;  // STANDARD
            if (occ == NB_OCC_EXTENDED || occ == NB_OCC_TWO_WAY) {
                // maps preceding the stencil that produce its input (back to the
                // previous stencil)
                for (int j = i - 1; j >= 0 && !is_stencil(c[j].op); --j)
                    if (c[j].op == NB_SK_AXPBY && c[j].y == c[i].x) split[j] = 1;
            }
            if (occ == NB_OCC_TWO_WAY) {
                // maps / reduces following the stencil that consume its output
                for (int j = i + 1; j < n && !is_stencil(c[j].op); ++j) {
                    if (c[j].op == NB_SK_SCALAR) continue;  // slots, not fields
                    const bool b_reads = c[j].b != 0.0 || c[j].b_slot >= 0;
                    const bool uses = c[j].x == c[i].y || (c[j].op == NB_SK_DOT && c[j].y == c[i].y) ||
                                      (c[j].op == NB_SK_AXPBY && b_reads && c[j].y == c[i].y);
                    if (uses) split[j] = 1;
                }
            }
        }
    }
    auto add = [&](Node nd) {
        nd.id = (int)P.nodes.size();
        P.nodes.push_back(nd);
        return nd.id;
    };
    auto accesses = [&](int i, nb_view v, bool fin) {
        std::vector<Access> a;
        const nb_container &k = c[i];
        const int m = view_mask(v);
        if (k.op == NB_SK_AXPBY) {
            a.push_back({k.x, m, false});
            if (k.b != 0.0 || k.b_slot >= 0) a.push_back({k.y, m, false});
            if (k.a_slot >= 0) a.push_back({SCALAR_BASE + k.a_slot, R_ALL, false});
            if (k.b_slot >= 0) a.push_back({SCALAR_BASE + k.b_slot, R_ALL, false});
            a.push_back({k.y, m, true});
        } else if (is_stencil(k.op)) {
            a.push_back({k.x, stencil_read_mask(v), false});
            a.push_back({k.y, m, true});
        } else if (k.op == NB_SK_SCALAR) {
            if (k.sop != NB_SC_SET) a.push_back({SCALAR_BASE + k.x, R_ALL, false});
            if (k.sop == NB_SC_DIV) a.push_back({SCALAR_BASE + k.y, R_ALL, false});
            a.push_back({SCALAR_BASE + k.slot, R_ALL, true});
        } else {
            a.push_back({k.x, m, false});
            a.push_back({k.y, m, false});
            a.push_back({TP_FIELD, R_ALL, true});  // shared partial / plane-sum scratch
            if (fin) a.push_back({SCALAR_BASE + k.slot, R_ALL, true});
        }
        return a;
    };
    static const char *kname[] = {"axpby", "laplace7", "dot", "poisson", "scalar", "lbm"};
    for (int i = 0; i < n; ++i) {
        auto mk = [&](nb_view v, bool fin) {
            Node nd;
            nd.op = c[i].op == NB_SK_AXPBY    ? SK_MAP
                    : is_stencil(c[i].op)      ? SK_STENCIL
                    : c[i].op == NB_SK_SCALAR ? SK_SCALAR
                                              : SK_REDUCE;
            nd.view = v;
            nd.container = i;
            nd.incoherent = incoh[i] != 0;
            nd.finalize = fin;
            nd.acc = accesses(i, v, fin);
            char buf[64];
            snprintf(buf, sizeof buf, "%s#%d%s", kname[c[i].op], i,
                     v == NB_VIEW_STANDARD ? "" : (v == NB_VIEW_INTERNAL ? "[int]" : "[bnd]"));
            nd.name = buf;
            return add(nd);
        };
        const bool red = c[i].op == NB_SK_DOT;
        if (!split[i]) {
            if (halo_before[i] >= 0) {
                Node h;
                h.op = SK_HALO;
                h.halo_field = halo_before[i];
                h.acc = {{halo_before[i], R_BLO | R_BHI, false}, {halo_before[i], R_HLO | R_HHI, true}};
                h.halo_lbm = c[i].op == NB_SK_LBM;
                h.name = "halo(f" + std::to_string(halo_before[i]) + ")";
                add(h);
            }
            mk(NB_VIEW_STANDARD, red);
            continue;
        }
        // split: the boundary part of a map first (its planes feed the halo),
        // then the internal part; stencils / reduces: internal, then boundary
        if (c[i].op == NB_SK_AXPBY) {
            mk(NB_VIEW_BOUNDARY, false);
            mk(NB_VIEW_INTERNAL, false);
        } else {
            if (halo_before[i] >= 0) {
                Node h;
                h.op = SK_HALO;
                h.halo_field = halo_before[i];
                h.acc = {{halo_before[i], R_BLO | R_BHI, false}, {halo_before[i], R_HLO | R_HHI, true}};
                h.halo_lbm = c[i].op == NB_SK_LBM;
                h.name = "halo(f" + std::to_string(halo_before[i]) + ")";
                add(h);
            }
            mk(NB_VIEW_INTERNAL, false);
            mk(NB_VIEW_BOUNDARY, red);  // a split reduce finalizes in its boundary part
        }
    }
    return NB_OK;
}

nb_status plan_graph(const nb_container *cin, int n, int nparts, nb_occ occ, Plan &P) {
    if (n < 0 || (n > 0 && !cin)) NB_FAIL(NB_EINVAL, "no containers");
    // normalised copy: a_slot / b_slot = -1 unless flagged
    std::vector<nb_container> cv(cin, cin + n);
    for (auto &k : cv) {
        if (!(k.flags & NB_SK_A_SLOT)) k.a_slot = -1;
        if (!(k.flags & NB_SK_B_SLOT)) k.b_slot = -1;
    }
    const nb_container *c = cv.data();
    if (nparts < 1) NB_FAIL(NB_EINVAL, "nparts < 1");
    if (occ < NB_OCC_NONE || occ > NB_OCC_TWO_WAY) NB_FAIL(NB_EINVAL, "bad OCC mode");
    NB_TRY(build_nodes(c, n, nparts, occ, P));
    const int N = (int)P.nodes.size();
    // A. data edges (sequential semantics), then the transitive reduction
    std::vector<std::vector<int>> adj(N);
    for (int j = 0; j < N; ++j)
        for (int i = 0; i < j; ++i)
            if (conflict(P.nodes[i], P.nodes[j])) adj[i].push_back(j);
    for (int i = 0; i < N; ++i) {
        std::vector<int> keep;
        for (int j : adj[i])
            if (!reaches(adj, i, j, j)) keep.push_back(j);
        adj[i] = keep;
    }
    for (int i = 0; i < N; ++i)
        for (int j : adj[i]) P.data.push_back({i, j});
    // B. hints: launch every internal node that is independent of a halo node
    // before it (otherwise the host enqueues the transfer first and nothing
    // overlaps, L318-L330)
    std::vector<std::vector<int>> both = adj;
    for (int h = 0; h < N; ++h) {
        if (P.nodes[h].op != SK_HALO) continue;
        for (int k = 0; k < N; ++k) {
            if (P.nodes[k].view != NB_VIEW_INTERNAL) continue;
            if (reaches(adj, k, h) || reaches(adj, h, k)) continue;  // not concurrent
            if (reaches(both, h, k)) continue;                       // would close a cycle
            P.hints.push_back({k, h});
            both[k].push_back(h);
        }
    }
    // C. levels, streams, events, order
    std::vector<int> level;
    std::vector<std::vector<int>> levels;
    if (!bfs_levels(N, P.data, level, levels)) NB_FAIL(NB_EINVAL, "dependency cycle");
    std::vector<std::vector<int>> parents(N);
    for (auto &e : P.data) parents[e.second].push_back(e.first);
    // compute nodes share the BFS-mapped streams; halo nodes get a stream of
    // their own (a transfer enqueued on a compute stream would queue behind
    // the very internal work it is meant to overlap with)
    int ncomp = 0;
    bool any_halo = false;
    for (auto &lv : levels) {
        int w = 0;
        for (int u : lv) {
            if (P.nodes[u].op == SK_HALO)
                any_halo = true;
            else
                ++w;
        }
        ncomp = std::max(ncomp, w);
    }
    ncomp = std::max(ncomp, 1);
    const int halo_stream = ncomp;
    P.nstreams = ncomp + (any_halo ? 1 : 0);
    for (auto &lv : levels) {
        std::vector<char> taken(P.nstreams, 0);
        std::vector<int> pending;
        for (int u : lv) {  // a parent's stream first (saves events)
            if (P.nodes[u].op == SK_HALO) {
                P.nodes[u].stream = halo_stream;
                continue;
            }
            int s = -1;
            for (int p : parents[u])
                if (P.nodes[p].stream != halo_stream && !taken[P.nodes[p].stream]) {
                    s = P.nodes[p].stream;
                    break;
                }
            if (s < 0) {
                pending.push_back(u);
                continue;
            }
            taken[s] = 1;
            P.nodes[u].stream = s;
        }
        for (int u : pending) {
            int s = 0;
            while (taken[s]) ++s;
            taken[s] = 1;
            P.nodes[u].stream = s;
        }
        for (int u : lv) P.nodes[u].level = level[u];
    }
    P.nevents = 0;
    for (auto &e : P.data) {
        Node &a = P.nodes[e.first], &b = P.nodes[e.second];
        if (a.stream == b.stream) continue;  // stream order suffices
        if (a.event < 0) a.event = P.nevents++;
        if (std::find(b.waits.begin(), b.waits.end(), a.event) == b.waits.end()) b.waits.push_back(a.event);
    }
    std::vector<std::pair<int, int>> all = P.data;
    all.insert(all.end(), P.hints.begin(), P.hints.end());
    std::vector<int> olevel;
    std::vector<std::vector<int>> olevels;
    if (!bfs_levels(N, all, olevel, olevels)) NB_FAIL(NB_EINVAL, "hint cycle");
    for (auto &lv : olevels)
        for (int u : lv) P.order.push_back(u);
    return NB_OK;
}

std::string plan_json(const Plan &P) {
    std::string s = "{\"nodes\":[";
    char buf[512];
    for (size_t i = 0; i < P.nodes.size(); ++i) {
        const Node &n = P.nodes[i];
        snprintf(buf, sizeof buf,
                 "%s{\"id\":%d,\"name\":\"%s\",\"op\":\"%s\",\"view\":\"%s\",\"container\":%d,\"incoherent\":%s,"
                 "\"finalize\":%s,\"level\":%d,\"stream\":%d,\"event\":%d,\"waits\":[",
                 i ? "," : "", n.id, n.name.c_str(), op_name(n.op), view_name(n.view), n.container,
                 n.incoherent ? "true" : "false", n.finalize ? "true" : "false", n.level, n.stream, n.event);
        s += buf;
        for (size_t k = 0; k < n.waits.size(); ++k) s += (k ? "," : "") + std::to_string(n.waits[k]);
        s += "]}";
    }
    auto pairs = [&](const char *key, const std::vector<std::pair<int, int>> &v) {
        s += std::string(",\"") + key + "\":[";
        for (size_t k = 0; k < v.size(); ++k)
            s += (k ? ",[" : "[") + std::to_string(v[k].first) + "," + std::to_string(v[k].second) + "]";
        s += "]";
    };
    s += "]";
    pairs("data", P.data);
    pairs("hints", P.hints);
    s += ",\"order\":[";
    for (size_t k = 0; k < P.order.size(); ++k) s += (k ? "," : "") + std::to_string(P.order[k]);
    s += "],\"streams\":" + std::to_string(P.nstreams) + ",\"events\":" + std::to_string(P.nevents) + "}";
    return s;
}

nb_status copy_out(const std::string &s, char *buf, int64_t cap, int64_t *len) {
    if (len) *len = (int64_t)s.size();
    if (!buf) return NB_OK;
    if (cap < (int64_t)s.size() + 1) NB_FAIL(NB_EINVAL, "buffer too small (%lld < %zu)", (long long)cap, s.size() + 1);
    memcpy(buf, s.c_str(), s.size() + 1);
    return NB_OK;
}

}  // namespace

// ===========================================================================
// C ABI
// ===========================================================================
extern "C" nb_status nb_skeleton_plan(int32_t nparts, nb_occ occ, const nb_container *containers, int32_t n,
                                      char *json, int64_t cap, int64_t *len) {
    Plan P;
    NB_TRY(plan_graph(containers, n, nparts, occ, P));
    return copy_out(plan_json(P), json, cap, len);
}

struct nb_skeleton {
    nb_grid *g = nullptr;
    nb_occ occ = NB_OCC_NONE;
    std::vector<nb_field *> fields;  // field id -> field
    std::vector<nb_container> cont;
    Plan plan;
    bool compiled = false;
    std::vector<cudaStream_t> streams;
    std::vector<cudaEvent_t> events;
    cudaEvent_t ev_start = nullptr;
    std::vector<cudaEvent_t> ev_end;
};

static int field_id(nb_skeleton *s, nb_field *f) {
    for (size_t i = 0; i < s->fields.size(); ++i)
        if (s->fields[i] == f) return (int)i;
    s->fields.push_back(f);
    return (int)s->fields.size() - 1;
}

extern "C" nb_status nb_skeleton_create(nb_grid *g, nb_occ occ, nb_skeleton **out) {
    if (!g || !out) NB_FAIL(NB_EINVAL, "nb_skeleton_create: NULL argument");
    if (occ < NB_OCC_NONE || occ > NB_OCC_TWO_WAY) NB_FAIL(NB_EINVAL, "bad OCC mode");
    if (g->sparse) NB_FAIL(NB_EUNSUPPORTED, "the Skeleton runs on dense grids");
    nb_skeleton *s = new nb_skeleton();
    s->g = g;
    s->occ = occ;
    g->nsolvers++;
    *out = s;
    return NB_OK;
}

static nb_status sk_push(nb_skeleton *s, const nb_container &c) {
    if (!s) NB_FAIL(NB_EINVAL, "NULL skeleton");
    if (s->compiled) NB_FAIL(NB_ESTATE, "skeleton already compiled");
    s->cont.push_back(c);
    return NB_OK;
}

static nb_status sk_add(nb_skeleton *s, int op, nb_field *x, nb_field *y, double a, double b, int slot,
                        int a_slot = -1, int b_slot = -1) {
    if (!s || !x || !y) NB_FAIL(NB_EINVAL, "NULL argument");
    if (x->g != s->g || y->g != s->g) NB_FAIL(NB_EMISMATCH, "field of another grid");
    if (x->dt != y->dt || x->card != y->card) NB_FAIL(NB_EMISMATCH, "dtype / cardinality mismatch");
    if ((op == NB_SK_LAPLACE7 || op == NB_SK_POISSON) && (x->card != 1 || x == y))
        NB_FAIL(NB_EINVAL, "7-point stencil: two distinct scalar fields");
    if ((a_slot >= 0 || b_slot >= 0) && x->dt != NB_F64) NB_FAIL(NB_EUNSUPPORTED, "device-scalar maps: fp64 fields");
    if (a_slot >= NB_DOT_SLOTS || b_slot >= NB_DOT_SLOTS) NB_FAIL(NB_EINVAL, "coefficient slot out of range");
    nb_container c;
    memset(&c, 0, sizeof c);
    c.op = op;
    c.x = field_id(s, x);
    c.y = field_id(s, y);
    c.a = a;
    c.b = b;
    c.slot = slot;
    c.a_slot = a_slot < 0 ? -1 : a_slot;
    c.b_slot = b_slot < 0 ? -1 : b_slot;
    c.flags = (a_slot >= 0 ? NB_SK_A_SLOT : 0) | (b_slot >= 0 ? NB_SK_B_SLOT : 0);
    return sk_push(s, c);
}

extern "C" nb_status nb_skeleton_axpby(nb_skeleton *s, double a, nb_field *x, double b, nb_field *y) {
    return sk_add(s, NB_SK_AXPBY, x, y, a, b, 0);
}
extern "C" nb_status nb_skeleton_axpby_s(nb_skeleton *s, double a, int32_t a_slot, nb_field *x, double b,
                                         int32_t b_slot, nb_field *y) {
    return sk_add(s, NB_SK_AXPBY, x, y, a, b, 0, a_slot, b_slot);
}
extern "C" nb_status nb_skeleton_laplace7(nb_skeleton *s, nb_field *x, nb_field *y) {
    return sk_add(s, NB_SK_LAPLACE7, x, y, 0.0, 0.0, 0);
}
extern "C" nb_status nb_skeleton_poisson(nb_skeleton *s, nb_field *x, nb_field *y) {
    return sk_add(s, NB_SK_POISSON, x, y, 0.0, 0.0, 0);
}
extern "C" nb_status nb_skeleton_dot(nb_skeleton *s, nb_field *x, nb_field *y, int32_t slot) {
    if (slot < 0 || slot >= NB_DOT_SLOTS) NB_FAIL(NB_EINVAL, "slot out of range [0, %d)", NB_DOT_SLOTS);
    return sk_add(s, NB_SK_DOT, x, y, 0.0, 0.0, slot);
}
extern "C" nb_status nb_skeleton_scalar(nb_skeleton *s, nb_scalar_op sop, int32_t in0, int32_t in1, int32_t out,
                                        double a) {
    if (sop < NB_SC_DIV || sop > NB_SC_SET) NB_FAIL(NB_EINVAL, "bad scalar op");
    for (int32_t v : {in0, in1, out})
        if (v < 0 || v >= NB_DOT_SLOTS) NB_FAIL(NB_EINVAL, "scalar slot out of range [0, %d)", NB_DOT_SLOTS);
    nb_container c;
    memset(&c, 0, sizeof c);
    c.op = NB_SK_SCALAR;
    c.sop = sop;
    c.x = in0;
    c.y = in1;
    c.slot = out;
    c.a = a;
    c.a_slot = c.b_slot = -1;
    return sk_push(s, c);
}
extern "C" nb_status nb_skeleton_lbm(nb_skeleton *s, nb_field *fin, nb_field *fout, const nb_lbm_params *prm) {
    if (!prm) NB_FAIL(NB_EINVAL, "NULL LBM parameters");
    if (!fin || !fout || fin->dt != NB_F32 || fin->card != Q19) NB_FAIL(NB_EMISMATCH, "LBM: fp32 fields of 19 components");
    if (prm->bc != NB_LBM_CAVITY) NB_FAIL(NB_EUNSUPPORTED, "Skeleton LBM containers: cavity boundaries");
    if (fin == fout) NB_FAIL(NB_EINVAL, "twoPop needs two distinct buffers");
    NB_TRY(sk_add(s, NB_SK_LBM, fin, fout, prm->omega, prm->u_lid, 0));
    s->cont.back().c = prm->rho_w;
    s->cont.back().sop = prm->bc;
    return NB_OK;
}

__global__ void k_sk_scalar(double *s, int sop, int x, int y, int out, double a) {
    if (threadIdx.x != 0) return;
    if (sop == NB_SC_DIV)
        s[out] = s[x] / s[y];
    else if (sop == NB_SC_COPY)
        s[out] = s[x];
    else
        s[out] = a;
}

extern "C" nb_status nb_skeleton_set_scalar(nb_skeleton *s, int32_t slot, double value) {
    if (!s) NB_FAIL(NB_EINVAL, "NULL skeleton");
    if (slot < 0 || slot >= NB_DOT_SLOTS) NB_FAIL(NB_EINVAL, "slot out of range");
    DeviceGuard dg(s->g->device);
    LaunchScope ls(s->g, s->g->cs, "k_sk_scalar");
    k_sk_scalar<<<1, 32, 0, s->g->cs>>>(s->g->dots, NB_SC_SET, 0, 0, slot, value);
    return nb_launch_check("k_sk_scalar");
}

// y = A x + B y with device-scalar coefficients (include/nb.h AXPBY rules)
enum { SKA_B1 = 0, SKA_A1 = 1, SKA_B0 = 2, SKA_GEN = 3 };
template <int MODE>
__global__ void __launch_bounds__(256) k_sk_axpby(const double *__restrict__ x, double *__restrict__ y, int64_t n,
                                                  double a, const double *as, double b, const double *bs) {
    const double A = as ? a * *as : a, B = bs ? b * *bs : b;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const double xv = x[i];
        if (MODE == SKA_B1)
            y[i] = fma(A, xv, y[i]);
        else if (MODE == SKA_A1)
            y[i] = fma(B, y[i], xv);
        else if (MODE == SKA_B0)
            y[i] = A * xv;
        else
            y[i] = fma(A, xv, B * y[i]);
    }
}

static nb_status sk_axpby_dev(nb_grid *g, const nb_container &c, const nb_field *x, nb_field *y, nb_view v,
                              cudaStream_t st) {
    const double *as = c.a_slot >= 0 ? g->dots + c.a_slot : nullptr;
    const double *bs = c.b_slot >= 0 ? g->dots + c.b_slot : nullptr;
    const int mode = (c.b_slot < 0 && c.b == 1.0)   ? SKA_B1
                     : (c.a_slot < 0 && c.a == 1.0) ? SKA_A1
                     : (c.b_slot < 0 && c.b == 0.0) ? SKA_B0
                                                    : SKA_GEN;
    for (int p = g->first_local; p < g->first_local + g->nlocal; ++p) {
        const int64_t cs = nb_cstride(x, p);
        for (auto rg : view_ranges(g, p, v))
            for (int k = 0; k < x->card; ++k) {
                const int64_t off = (int64_t)k * cs + (int64_t)(rg.first + 1) * x->ps;
                const int64_t n = (int64_t)(rg.second - rg.first) * x->ps;
                const double *xp = (const double *)x->base[p] + off;
                double *yp = (double *)y->base[p] + off;
                const int blocks = (int)std::min<int64_t>((n + 255) / 256, 148 * 8);
                LaunchScope ls(g, st, "k_sk_axpby");
                if (mode == SKA_B1)
                    k_sk_axpby<SKA_B1><<<blocks, 256, 0, st>>>(xp, yp, n, c.a, as, c.b, bs);
                else if (mode == SKA_A1)
                    k_sk_axpby<SKA_A1><<<blocks, 256, 0, st>>>(xp, yp, n, c.a, as, c.b, bs);
                else if (mode == SKA_B0)
                    k_sk_axpby<SKA_B0><<<blocks, 256, 0, st>>>(xp, yp, n, c.a, as, c.b, bs);
                else
                    k_sk_axpby<SKA_GEN><<<blocks, 256, 0, st>>>(xp, yp, n, c.a, as, c.b, bs);
                NB_TRY(nb_launch_check("k_sk_axpby"));
            }
    }
    return NB_OK;
}

extern "C" nb_status nb_skeleton_compile(nb_skeleton *s) {
    if (!s) NB_FAIL(NB_EINVAL, "NULL skeleton");
    if (s->compiled) return NB_OK;
    NB_TRY(plan_graph(s->cont.data(), (int)s->cont.size(), s->g->nparts, s->occ, s->plan));
    DeviceGuard dg(s->g->device);
    s->streams.resize(std::max(s->plan.nstreams, 1));
    for (auto &st : s->streams) NB_CUDA(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
    s->events.resize(s->plan.nevents);
    for (auto &e : s->events) NB_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    NB_CUDA(cudaEventCreateWithFlags(&s->ev_start, cudaEventDisableTiming));
    s->ev_end.resize(s->streams.size());
    for (auto &e : s->ev_end) NB_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    s->compiled = true;
    return NB_OK;
}

// run one node on stream st (the library ops enqueue on g->cs: point it at st)
static nb_status run_node(nb_skeleton *s, const Node &n, cudaStream_t st) {
    nb_grid *g = s->g;
    cudaStream_t saved = g->cs;
    g->cs = st;
    nb_status r = NB_OK;
    if (n.op == SK_HALO) {
        nb_field *f = s->fields[n.halo_field];
        r = n.halo_lbm ? nb_halo_run(f, false, 9, 14, 14, 19, st)  // the z-crossing populations
                       : nb_halo_exchange_planes(f, 0, f->card, true, true, st);
    } else {
        const nb_container &c = s->cont[n.container];
        if (c.op == NB_SK_SCALAR) {
            LaunchScope ls(g, st, "k_sk_scalar");
            k_sk_scalar<<<1, 32, 0, st>>>(g->dots, c.sop, c.x, c.y, c.slot, c.a);
            r = nb_launch_check("k_sk_scalar");
            g->cs = saved;
            return r;
        }
        nb_field *x = s->fields[c.x], *y = s->fields[c.y];
        if (c.op == NB_SK_AXPBY) {
            r = (c.a_slot >= 0 || c.b_slot >= 0) ? sk_axpby_dev(g, c, x, y, n.view, st) : nb_axpby(c.a, x, c.b, y, n.view);
        } else if (c.op == NB_SK_LAPLACE7 || c.op == NB_SK_POISSON) {
            r = nb_stencil7(x, y, n.view, c.op == NB_SK_POISSON);
        } else if (c.op == NB_SK_LBM) {
            nb_lbm_params prm;
            prm.omega = c.a;
            prm.u_lid = c.b;
            prm.rho_w = c.c;
            prm.bc = (nb_lbm_bc)c.sop;
            r = nb_lbm_view(x, y, &prm, n.view);
        } else {
            r = nb_dot_partials_view(x, y, n.view);
            if (r == NB_OK && n.finalize) r = nb_reduce_finalize(g, x->card, FIN_STORE, nullptr, c.slot);
        }
    }
    g->cs = saved;
    return r;
}

extern "C" nb_status nb_skeleton_run(nb_skeleton *s) {
    NB_RANGE("nb_skeleton_run");
    if (!s) NB_FAIL(NB_EINVAL, "NULL skeleton");
    NB_TRY(nb_skeleton_compile(s));
    nb_grid *g = s->g;
    DeviceGuard dg(g->device);
    // everything before the run (uploads, fills) is ordered on the compute stream
    NB_CUDA(cudaEventRecord(s->ev_start, g->cs));
    for (auto st : s->streams) NB_CUDA(cudaStreamWaitEvent(st, s->ev_start, 0));
    for (int u : s->plan.order) {
        const Node &n = s->plan.nodes[u];
        cudaStream_t st = s->streams[n.stream];
        for (int e : n.waits) NB_CUDA(cudaStreamWaitEvent(st, s->events[e], 0));
        NB_TRY(run_node(s, n, st));
        if (n.event >= 0) NB_CUDA(cudaEventRecord(s->events[n.event], st));
    }
    // join: later work on the compute stream sees every result
    for (size_t i = 0; i < s->streams.size(); ++i) {
        NB_CUDA(cudaEventRecord(s->ev_end[i], s->streams[i]));
        NB_CUDA(cudaStreamWaitEvent(g->cs, s->ev_end[i], 0));
    }
    return NB_OK;
}

extern "C" nb_status nb_skeleton_result(nb_skeleton *s, int32_t slot, double *host) {
    if (!s || !host) NB_FAIL(NB_EINVAL, "NULL argument");
    if (slot < 0 || slot >= NB_DOT_SLOTS) NB_FAIL(NB_EINVAL, "slot out of range");
    DeviceGuard dg(s->g->device);
    NB_CUDA(cudaMemcpyAsync(host, s->g->dots + slot, sizeof(double), cudaMemcpyDeviceToHost, s->g->cs));
    NB_CUDA(cudaStreamSynchronize(s->g->cs));
    return NB_OK;
}

extern "C" nb_status nb_skeleton_describe(nb_skeleton *s, char *json, int64_t cap, int64_t *len) {
    if (!s) NB_FAIL(NB_EINVAL, "NULL skeleton");
    if (!s->compiled) {  // plan only (no streams yet)
        Plan P;
        NB_TRY(plan_graph(s->cont.data(), (int)s->cont.size(), s->g->nparts, s->occ, P));
        return copy_out(plan_json(P), json, cap, len);
    }
    return copy_out(plan_json(s->plan), json, cap, len);
}

extern "C" nb_status nb_skeleton_destroy(nb_skeleton *s) {
    if (!s) return NB_OK;
    DeviceGuard dg(s->g->device);
    for (auto st : s->streams) {
        cudaStreamSynchronize(st);
        cudaStreamDestroy(st);
    }
    for (auto e : s->events) cudaEventDestroy(e);
    for (auto e : s->ev_end) cudaEventDestroy(e);
    if (s->ev_start) cudaEventDestroy(s->ev_start);
    s->g->nsolvers--;
    delete s;
    return NB_OK;
}
