// ug_selector.cpp -- schedule selection when parallel_info is absent.
//
// The paper trains LightGBM on Table 7's features.  This build has three
// tiers, consulted in order:
//  1. a table of schedules MEASURED on B200 for the named configs (scripts/sweep.py writes
//     selector_table.json), keyed by the Table 7 features plus the feature width F that Fig. 7
//     shows matters: op class, F, mean in-degree, degree CV (= std_nnz /
//     mean), V -- among the entries whose ranges hold the graph, the nearest (log distance
//     to the range centres) wins;
//  2. a learned model (selector_model.txt, scripts/train_selector.py): per op class a
//     cost-sensitive regression tree trained on a synthetic B200 corpus of graphs
//     (scripts/selector_corpus.py), features log2 V, log2 E, log2 mean degree, CV,
//     log2(max degree / mean), log2 F; each leaf names the schedule with the lowest mean
//     log-slowdown of its training points;
//  3. priors (Table 9's observations, re-derived for B200 in DESIGN.md).
// Each lookup is a linear scan / a tree walk of a few nodes: far under the paper's 0.2 ms
// budget.
#include <dlfcn.h>

#include <algorithm>
#include <cmath>
#include <cctype>
#include <cstdlib>
#include <cstring>
#include <fstream>
#include <mutex>
#include <sstream>
#include <string>
#include <vector>

#include "ug_internal.h"
#include "ug_runtime.h"

namespace ug {

struct Entry {
    int op_class = -1;          // -1 = any
    double F_lo = 0, F_hi = 1e18, deg_lo = 0, deg_hi = 1e18, cv_lo = 0, cv_hi = 1e18, V_lo = 0, V_hi = 1e18;
    ug_schedule sched{};
};

static std::mutex g_mu;
static std::vector<Entry> g_table;
static bool g_loaded = false;

// Learned model: one tree per op class (index = class_of()).
struct Node {
    int feature = -1;       // -1: leaf
    double thr = 0;
    int left = -1, right = -1;
    ug_schedule sched{};
};
static std::vector<Node> g_trees[6];
static bool g_model_loaded = false;

// Learned model, nearest-neighbour form (round 2): per op class the corpus points themselves --
// standardised, weighted features and the log-slowdown of every candidate schedule at that
// point.  A query takes its k nearest corpus graphs, averages their log-slowdown vectors with
// weights 1 / (distance + 1e-3), and picks the schedule with the lowest average.  Used for the
// classes where leave-graphs-out CV favours it over the tree (scripts/train_selector.py).
struct Knn {
    int k = 0;
    double w[6] = {}, mu[6] = {}, sd[6] = {};
    std::vector<ug_schedule> scheds;
    std::vector<std::vector<double>> X;     // [n][6] standardised * weighted
    std::vector<std::vector<float>> Y;      // [n][n_sched] log-slowdown
};
static Knn g_knn[6];

static int class_of(const std::string &s) {
    if (s == "msg") return 0;
    if (s == "agg") return 1;
    if (s == "dot_msg") return 2;
    if (s == "dot_agg") return 3;
    if (s == "agg_bin") return 4;   // aggregation with two operands (e.g. u_mul_e_sum)
    if (s == "agg_ext") return 5;   // max / min aggregation
    return -1;
}

// Minimal JSON reader for {"entries": [{"key": number | "string", ...}, ...]}.
static bool parse_table(const std::string &txt, std::vector<Entry> *out, std::string *why) {
    size_t p = txt.find("\"entries\"");
    if (p == std::string::npos) { *why = "no \"entries\" key"; return false; }
    p = txt.find('[', p);
    if (p == std::string::npos) { *why = "entries is not an array"; return false; }
    std::vector<Entry> res;
    while (true) {
        size_t ob = txt.find_first_of("{]", p + 1);
        if (ob == std::string::npos) { *why = "unterminated entries"; return false; }
        if (txt[ob] == ']') break;
        size_t cb = txt.find('}', ob);
        if (cb == std::string::npos) { *why = "unterminated object"; return false; }
        std::string obj = txt.substr(ob + 1, cb - ob - 1);
        Entry e;
        size_t q = 0;
        while ((q = obj.find('"', q)) != std::string::npos) {
            size_t qe = obj.find('"', q + 1);
            if (qe == std::string::npos) break;
            std::string key = obj.substr(q + 1, qe - q - 1);
            size_t colon = obj.find(':', qe);
            if (colon == std::string::npos) break;
            size_t vs = colon + 1;
            while (vs < obj.size() && std::isspace((unsigned char)obj[vs])) ++vs;
            std::string sval;
            double nval = 0;
            bool is_str = vs < obj.size() && obj[vs] == '"';
            size_t ve;
            if (is_str) {
                ve = obj.find('"', vs + 1);
                sval = obj.substr(vs + 1, ve - vs - 1);
                ++ve;
            } else {
                ve = obj.find_first_of(",}", vs);
                if (ve == std::string::npos) ve = obj.size();
                nval = std::strtod(obj.substr(vs, ve - vs).c_str(), nullptr);
            }
            if (key == "class") e.op_class = class_of(sval);
            else if (key == "F_lo") e.F_lo = nval;
            else if (key == "F_hi") e.F_hi = nval;
            else if (key == "deg_lo") e.deg_lo = nval;
            else if (key == "deg_hi") e.deg_hi = nval;
            else if (key == "cv_lo") e.cv_lo = nval;
            else if (key == "cv_hi") e.cv_hi = nval;
            else if (key == "V_lo") e.V_lo = nval;
            else if (key == "V_hi") e.V_hi = nval;
            else if (key == "schedule") {
                if (ug_schedule_parse(sval.c_str(), &e.sched) != UG_OK) { *why = "bad schedule " + sval; return false; }
            }
            q = ve;
        }
        if (e.sched.strategy != UG_SCHED_AUTO) res.push_back(e);
        p = cb;
    }
    *out = std::move(res);
    return true;
}

static std::string default_table_path() {
    const char *env = std::getenv("UG_SELECTOR_TABLE");
    if (env && *env) return env;
    Dl_info info;
    if (dladdr((void *)&default_table_path, &info) && info.dli_fname) {
        std::string f(info.dli_fname);
        size_t sl = f.rfind('/');
        return (sl == std::string::npos ? std::string(".") : f.substr(0, sl)) + "/selector_table.json";
    }
    return "selector_table.json";
}

static ug_status load_file(const std::string &path, bool quiet) {
    std::ifstream in(path);
    if (!in) return quiet ? UG_OK : set_error(UG_ERR_INVALID_ARG, "cannot open " + path);
    std::stringstream ss;
    ss << in.rdbuf();
    std::vector<Entry> t;
    std::string why;
    if (!parse_table(ss.str(), &t, &why)) return set_error(UG_ERR_INVALID_ARG, "selector table " + path + ": " + why);
    g_table = std::move(t);
    return UG_OK;
}

static std::string default_model_path() {
    const char *env = std::getenv("UG_SELECTOR_MODEL");
    if (env) return env;   // "" disables the model
    std::string t = default_table_path();
    size_t sl = t.rfind('/');
    return (sl == std::string::npos ? std::string(".") : t.substr(0, sl)) + "/selector_model.txt";
}

// Text format of scripts/train_selector.py: "class <name> <n>" then n lines
// "<id> <feature> <threshold> <left> <right> <schedule|->"; '#' lines are comments.
// Nearest-neighbour block: "knn <class> <k> <npoints> <nsched>", then lines "w ...", "mu ...",
// "sd ..." (6 numbers each), "s <schedule> x nsched", and npoints lines "p <6 features> <nsched
// log-slowdowns>".
static ug_status load_knn(std::ifstream &in, std::istringstream &head, const std::string &path, Knn *out,
                          int *cls_out) {
    std::string name;
    int k = 0, n = 0, ns = 0;
    if (!(head >> name >> k >> n >> ns) || k <= 0 || n <= 0 || ns <= 0)
        return set_error(UG_ERR_INVALID_ARG, "selector model " + path + ": bad knn header");
    const int cls = class_of(name);
    if (cls < 0) return set_error(UG_ERR_INVALID_ARG, "selector model: unknown class " + name);
    Knn m;
    m.k = k;
    std::string line, tag;
    for (double *arr : {m.w, m.mu, m.sd}) {
        if (!std::getline(in, line)) return set_error(UG_ERR_INVALID_ARG, "selector model: truncated knn");
        std::istringstream ls(line);
        ls >> tag;
        for (int i = 0; i < 6; ++i)
            if (!(ls >> arr[i])) return set_error(UG_ERR_INVALID_ARG, "selector model: bad knn vector " + tag);
    }
    if (!std::getline(in, line)) return set_error(UG_ERR_INVALID_ARG, "selector model: truncated knn");
    {
        std::istringstream ls(line);
        ls >> tag;
        std::string sname;
        for (int i = 0; i < ns; ++i) {
            ug_schedule sc{};
            if (!(ls >> sname) || ug_schedule_parse(sname.c_str(), &sc) != UG_OK)
                return set_error(UG_ERR_INVALID_ARG, "selector model: bad knn schedule list");
            m.scheds.push_back(sc);
        }
    }
    for (int p = 0; p < n; ++p) {
        if (!std::getline(in, line)) return set_error(UG_ERR_INVALID_ARG, "selector model: truncated knn points");
        std::istringstream ls(line);
        ls >> tag;
        std::vector<double> x(6);
        std::vector<float> y(ns);
        for (int i = 0; i < 6; ++i)
            if (!(ls >> x[i])) return set_error(UG_ERR_INVALID_ARG, "selector model: bad knn point");
        for (int i = 0; i < ns; ++i)
            if (!(ls >> y[i])) return set_error(UG_ERR_INVALID_ARG, "selector model: bad knn point");
        m.X.push_back(std::move(x));
        m.Y.push_back(std::move(y));
    }
    *out = std::move(m);
    *cls_out = cls;
    return UG_OK;
}

static ug_status load_model(const std::string &path, bool quiet) {
    std::ifstream in(path);
    if (!in) return quiet ? UG_OK : set_error(UG_ERR_INVALID_ARG, "cannot open " + path);
    std::vector<Node> trees[6];
    Knn knns[6];
    std::string line;
    int cls = -1, remaining = 0;
    while (std::getline(in, line)) {
        if (line.empty() || line[0] == '#') continue;
        std::istringstream ls(line);
        if (remaining == 0) {
            std::string kw, name;
            if (line.compare(0, 4, "knn ") == 0) {
                ls >> kw;
                int kc = -1;
                Knn m;
                ug_status st = load_knn(in, ls, path, &m, &kc);
                if (st != UG_OK) return st;
                knns[kc] = std::move(m);
                continue;
            }
            int n = 0;
            if (!(ls >> kw >> name >> n) || kw != "class" || n <= 0)
                return set_error(UG_ERR_INVALID_ARG, "selector model " + path + ": bad class line: " + line);
            cls = class_of(name);
            if (cls < 0) return set_error(UG_ERR_INVALID_ARG, "selector model: unknown class " + name);
            trees[cls].assign(n, Node{});
            remaining = n;
            continue;
        }
        int id, f, l, r;
        double thr;
        std::string sched;
        if (!(ls >> id >> f >> thr >> l >> r >> sched) || id < 0 || id >= (int)trees[cls].size())
            return set_error(UG_ERR_INVALID_ARG, "selector model " + path + ": bad node line: " + line);
        Node &nd = trees[cls][id];
        nd.feature = f;
        nd.thr = thr;
        nd.left = l;
        nd.right = r;
        if (f < 0 && ug_schedule_parse(sched.c_str(), &nd.sched) != UG_OK)
            return set_error(UG_ERR_INVALID_ARG, "selector model: bad schedule " + sched);
        if (f >= 6 || (f >= 0 && (l < 0 || r < 0 || l >= (int)trees[cls].size() || r >= (int)trees[cls].size())))
            return set_error(UG_ERR_INVALID_ARG, "selector model: bad node " + std::to_string(id));
        --remaining;
    }
    if (remaining) return set_error(UG_ERR_INVALID_ARG, "selector model " + path + ": truncated");
    for (int c = 0; c < 6; ++c) {
        g_trees[c] = std::move(trees[c]);
        g_knn[c] = std::move(knns[c]);
    }
    return UG_OK;
}

static ug_schedule adapt(const Lowered &lw, ug_schedule s);

// k nearest corpus graphs, distance-weighted mean log-slowdown per schedule, best first
static std::vector<ug_schedule> knn_rank(const Knn &m, const double (&x)[6]) {
    double z[6];
    for (int i = 0; i < 6; ++i) z[i] = (x[i] - m.mu[i]) / m.sd[i] * m.w[i];
    std::vector<std::pair<double, int>> d(m.X.size());
    for (size_t p = 0; p < m.X.size(); ++p) {
        double s = 0;
        for (int i = 0; i < 6; ++i) s += (z[i] - m.X[p][i]) * (z[i] - m.X[p][i]);
        d[p] = {std::sqrt(s), (int)p};
    }
    const size_t k = std::min<size_t>((size_t)m.k, d.size());
    std::partial_sort(d.begin(), d.begin() + k, d.end());
    std::vector<std::pair<double, int>> score(m.scheds.size());
    for (size_t j = 0; j < m.scheds.size(); ++j) score[j] = {0.0, (int)j};
    double wsum = 0;
    for (size_t q = 0; q < k; ++q) {
        const double wt = 1.0 / (d[q].first + 1e-3);
        wsum += wt;
        for (size_t j = 0; j < m.scheds.size(); ++j) score[j].first += wt * m.Y[d[q].second][j];
    }
    std::sort(score.begin(), score.end());
    std::vector<ug_schedule> out;
    for (auto &sc : score) out.push_back(m.scheds[sc.second]);
    (void)wsum;
    return out;
}

static bool model_select(const ug_graph *g, const Lowered &lw, ug_schedule *out) {
    const std::vector<Node> &t = g_trees[lw.op_class];
    const Knn &m = g_knn[lw.op_class];
    if ((t.empty() && m.k == 0) || g->V <= 0 || g->E <= 0) return false;
    const double mean = std::max(g->mean_deg, 1e-9);
    const double x[6] = {std::log2((double)g->V), std::log2((double)g->E), std::log2(mean), g->std_nnz / mean,
                         std::log2(std::max<double>(1.0, (double)g->max_deg) / mean), std::log2((double)lw.args.F)};
    if (m.k > 0) {
        // the best-ranked schedule that resolves on this operator's layout
        for (const ug_schedule &sc : knn_rank(m, x)) {
            ug_schedule s2 = adapt(lw, sc);
            LaunchCfg cfg;
            if (resolve(g, lw, s2, &cfg) == UG_OK) { *out = s2; return true; }
        }
        return false;
    }
    int n = 0;
    for (int steps = 0; steps < 64 && t[n].feature >= 0; ++steps) n = x[t[n].feature] <= t[n].thr ? t[n].left : t[n].right;
    if (t[n].feature >= 0) return false;
    *out = t[n].sched;
    return true;
}

// A measured schedule applied to this operator's layout: drop a forced vector width the
// layout cannot take; an SV column tile may need more than 32 lanes at this layout's vector
// width (measured with float4 rows, applied to float2 rows): keep 32 lanes.
static ug_schedule adapt(const Lowered &lw, ug_schedule s) {
    if (s.vec > lw.max_vec) s.vec = 0;
    // edge lanes hold at most 8 feature vectors per lane: a wider row (or a narrower vector width
    // at this layout) takes the feature-lane warp-vertex kernel instead
    if ((s.flags & UG_SCHED_EDGELANES) &&
        (lw.dot || (lw.to_edges ? lw.args.W > 8 : (lw.args.W + lw.max_vec - 1) / lw.max_vec > 8)))
        s.flags &= ~UG_SCHED_EDGELANES;
    // (dot under SV with a column tile is k_dott, which picks its own vector width and packs P;
    // staged SV fixes vec = ftile / 32 itself)
    if (s.strategy == UG_SV && s.ftile > 0 && !lw.dot && !(s.flags & (UG_SCHED_TMA | UG_SCHED_ASYNC))) {
        const bool pack = (s.flags & UG_SCHED_PACK) && lw.pack_ok;
        const int vec = std::max(1, std::min(pack ? 4 : lw.a_vec, lw.b_vec));
        if (s.ftile / vec > 32 || s.ftile % vec) s.ftile = 32 * vec;
    }
    return s;
}

// Priors used when no measured entry matches.
static ug_schedule prior(const ug_graph *g, const Lowered &lw) {
    ug_schedule s{};
    const int W = lw.args.W, vec = lw.max_vec;
    const int chunks = (W + vec - 1) / vec;
    int lanes = 1;
    while (lanes < chunks && lanes < 32) lanes <<= 1;
    if (lw.op_class == 0) {            // message creation: thread-edge (Table 9: always TE)
        s.strategy = UG_TE; s.group = 1; s.tile = lanes;
    } else if (lw.op_class == 2 || lw.op_class == 3) {
        const Operand &A = lw.args.A, &B = lw.args.B;
        const bool uv = A.div == 1 && B.div == 1 &&
                        ((A.type == UG_T_SRC_V && B.type == UG_T_DST_V) || (A.type == UG_T_DST_V && B.type == UG_T_SRC_V));
        if (uv && lw.args.D >= 256) {                 // wide heads: column-tiled k_dott (r2 sweep, C5)
            s.strategy = UG_SV; s.group = 512; s.ftile = 128;
        } else if (lw.op_class == 2) {                // SDDMM: lanes over the head's D features
            int dl = 1;
            const int dch = (lw.args.D + vec - 1) / vec;
            while (dl < dch && dl < 32) dl <<= 1;
            s.strategy = UG_TE; s.group = 1; s.tile = dl;
        } else {
            s.strategy = UG_WV; s.group = 1; s.tile = 1;
        }
    } else {                           // aggregation (classes 1, 4, 5)
        if (W >= 32 || g->max_deg > 256) {
            s.strategy = UG_SV; s.group = 512; s.ftile = 0;
            if (W >= 256 && lw.pack_ok) s.flags = UG_SCHED_PACK;   // wide rows: aligned L2 slabs
        }
        else { s.strategy = UG_WV; s.group = 1; s.tile = 1; }
    }
    return s;
}

ug_status select_schedule(const ug_graph *g, const Lowered &lw, ug_schedule *out) {
    const char *force = std::getenv("UG_FORCE_SCHEDULE");
    if (force && *force) return ug_schedule_parse(force, out);
    std::lock_guard<std::mutex> lock(g_mu);
    if (!g_loaded) {
        g_loaded = true;
        load_file(default_table_path(), true);
    }
    if (!g_model_loaded) {
        g_model_loaded = true;
        const std::string mp = default_model_path();
        if (!mp.empty()) load_model(mp, true);
    }
    const double F = lw.args.F, deg = g->mean_deg, V = (double)g->V;
    const double cv = g->mean_deg > 0 ? g->std_nnz / g->mean_deg : 0.0;
    // 1. measured table: exact class first, then the parent class (agg_bin / agg_ext -> agg)
    const int classes[2] = {lw.op_class, (lw.op_class == 4 || lw.op_class == 5) ? 1 : -2};
    for (int pass = 0; pass < 2; ++pass) {
        if (classes[pass] == -2) break;
        // among the entries whose box holds the graph, the nearest one wins: distance = sum over
        // (F, mean degree, CV, V) of |log(x / geometric centre of the entry's range)| (boxes of
        // neighbouring configs overlap, e.g. C3 and C4 share F = 128 and mean degree ~7-8)
        const Entry *best = nullptr;
        double best_d = 0;
        auto ld = [](double x, double lo, double hi) {
            if (lo <= 0 || hi >= 1e17) return 0.0;     // open range: no preference
            return std::fabs(std::log(std::max(x, 1e-12) / std::sqrt(lo * hi)));
        };
        for (const Entry &e : g_table) {
            if (e.op_class != -1 && e.op_class != classes[pass]) continue;
            if (F < e.F_lo || F > e.F_hi || deg < e.deg_lo || deg > e.deg_hi || cv < e.cv_lo || cv > e.cv_hi ||
                V < e.V_lo || V > e.V_hi)
                continue;
            const double d = ld(F, e.F_lo, e.F_hi) + ld(deg, e.deg_lo, e.deg_hi) + ld(cv, e.cv_lo, e.cv_hi) +
                             ld(V, e.V_lo, e.V_hi);
            if (!best || d < best_d) { best = &e; best_d = d; }
        }
        if (best) {
            // a measured schedule that does not resolve on this operator's layout falls through
            // to the next tier
            ug_schedule s2 = adapt(lw, best->sched);
            LaunchCfg cfg;
            if (resolve(g, lw, s2, &cfg) == UG_OK) {
                *out = s2;
                return UG_OK;
            }
        }
        if (pass == 0) {
            // 2. learned model of the exact class (only if its pick resolves on this layout)
            ug_schedule s;
            LaunchCfg cfg;
            if (model_select(g, lw, &s)) {
                s = adapt(lw, s);
                if (resolve(g, lw, s, &cfg) == UG_OK) {
                    *out = s;
                    return UG_OK;
                }
            }
        }
    }
    // 3. priors
    *out = prior(g, lw);
    return UG_OK;
}

}  // namespace ug

extern "C" ug_status ug_schedule_select(const ug_graph *g, const ug_op_info *op, ug_schedule *out) {
    if (!out) return ug::set_error(UG_ERR_INVALID_ARG, "NULL out");
    ug::Lowered lw;
    ug_status st = ug::lower(g, op, &lw);
    if (st != UG_OK) return st;
    return ug::select_schedule(g, lw, out);
}

extern "C" ug_status ug_selector_load_model(const char *path) {
    if (!path) return ug::set_error(UG_ERR_INVALID_ARG, "NULL path");
    std::lock_guard<std::mutex> lock(ug::g_mu);
    ug::g_model_loaded = true;
    if (!*path) {                       // "" unloads the model
        for (auto &t : ug::g_trees) t.clear();
        for (auto &m : ug::g_knn) m = ug::Knn{};
        return UG_OK;
    }
    return ug::load_model(path, false);
}

extern "C" ug_status ug_selector_load(const char *path) {
    if (!path) return ug::set_error(UG_ERR_INVALID_ARG, "NULL path");
    std::lock_guard<std::mutex> lock(ug::g_mu);
    ug::g_loaded = true;
    return ug::load_file(path, false);
}
