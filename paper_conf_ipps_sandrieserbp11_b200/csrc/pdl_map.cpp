// pdl_map.cpp -- task decomposition and BLOCK mapping of tile tasks onto the
// execution group's Workers.
//
// PAPER.md SS IV-A: distribution specifiers "hold references to input and
// output parameter data-distributions (e.g., block, cyclic, block-cyclic) and
// optional sizes ... for possible data-decomposition of data-parallel tasks"
// (L1200-1208); example `(A:BLOCK:N, B:BLOCK:N)` (L1155-1156).  SS IV-B:
// "From that generic model a compiler or run-time can further automatically
// derive optimized mapping decisions to physical hardware elements"
// (L1262-1266).  Readings R4-R6: C is cut into ceil(M/tile) x
// ceil(N/tile) tile tasks; BLOCK distributes task rows / columns over a
// Gr x Gc Worker grid; the Worker grid minimises exchanged operand bytes.
#include <algorithm>
#include <cctype>
#include <cmath>
#include <cstdlib>
#include <limits>
#include <map>
#include <sstream>

#include "pdl_model.hpp"

namespace pdl {

static int64_t cdiv(int64_t a, int64_t b) { return b ? (a + b - 1) / b : 0; }

Rect Plan::rect(int w) const {
    if (!wrect.empty()) return wrect[w];
    int r = w / Gc, c = w % Gc;
    return Rect{row[r], row[r + 1], col[c], col[c + 1]};
}

// A row-panel of Worker (r,c) split in Gc chunks of qa rows (ceil): chunk j =
// panel rows [j*qa, min((j+1)*qa, rows)).  Gathering Gc chunks of qa rows
// each leaves the panel contiguous in the first `rows` rows of the buffer.
int64_t Plan::qa(int w) const {
    Rect R = rect(w);
    return cdiv(R.row1 - R.row0, Gc);
}

int64_t Plan::qb() const { return cdiv(K, Gr); }

double Plan::exchanged_elems() const {
    double tot = 0;
    for (int w = 0; w < G; ++w) {
        Rect R = rect(w);
        double rows = double(R.row1 - R.row0), cols = double(R.col1 - R.col0);
        tot += rows * K * (1.0 - 1.0 / Gc) + double(K) * cols * (1.0 - 1.0 / Gr);
    }
    return tot;
}

bool parse_dist(const char *s, DistSpec *out) {
    DistSpec d;
    if (!s) {
        *out = d;
        return true;
    }
    std::string v;
    for (const char *c = s; *c; ++c) v += (char)std::toupper((unsigned char)*c);
    std::string name = v, size;
    size_t colon = v.find(':');
    if (colon != std::string::npos) {
        name = v.substr(0, colon);
        size = v.substr(colon + 1);
    }
    for (auto &ch : name)
        if (ch == '_') ch = '-';
    if (name == "BLOCK") {
        d.kind = Dist::Block;   // BLOCK:N -- N (L1155) is the element count, implied by the task
    } else if (name == "DYNAMIC" && size.empty()) {
        d.kind = Dist::Dynamic;
    } else if (name == "CYCLIC" || name == "BLOCK-CYCLIC") {
        d.kind = name == "CYCLIC" ? Dist::Cyclic : Dist::BlockCyclic;
        d.b = 1;
        if (!size.empty() && name == "BLOCK-CYCLIC") {
            char *end = nullptr;
            long long b = std::strtoll(size.c_str(), &end, 10);
            if (!end || *end || b < 1) return false;
            d.b = b;
        }
    } else {
        return false;
    }
    *out = d;
    return true;
}

// Element segments of grid index g (of Gx) over T tasks of edge `tile` along a
// dimension of length L, merged when adjacent.
static std::vector<Seg> segs_of(const Plan &p, int g, int Gx, int64_t T, int64_t L, const std::vector<int64_t> &bnd) {
    std::vector<Seg> out;
    if (p.dist.kind == Dist::Block) {
        if (bnd[g + 1] > bnd[g]) out.push_back(Seg{bnd[g], bnd[g + 1]});
        return out;
    }
    const int64_t edge = p.tile ? p.tile : 1;
    const int64_t b = p.dist.b;
    for (int64_t q = g; q * b < T; q += Gx) {
        const int64_t lo = std::min(q * b * edge, L), hi = std::min((q + 1) * b * edge, L);
        if (hi <= lo) continue;
        if (!out.empty() && out.back().hi == lo) out.back().hi = hi;
        else out.push_back(Seg{lo, hi});
    }
    return out;
}

std::vector<Seg> Plan::row_segs(int r) const { return segs_of(*this, r, Gr, Tm, M, row); }
std::vector<Seg> Plan::col_segs(int c) const { return segs_of(*this, c, Gc, Tn, N, col); }

std::vector<double> worker_speeds(const Model &m, const std::vector<int> &workers) {
    std::vector<double> s;
    for (int w : workers) {
        double v = 1.0;
        if (const Property *p = m.prop(w, "RELATIVE_SPEED")) {
            char *end = nullptr;
            double x = std::strtod(p->value.c_str(), &end);
            if (end && !*end && x > 0 && std::isfinite(x)) v = x;
        }
        s.push_back(v);
    }
    return s;
}

Plan make_plan(int64_t M, int64_t N, int64_t K, int64_t tile, int G, DistSpec dist, const std::vector<double> *speeds) {
    Plan p;
    p.M = M; p.N = N; p.K = K; p.G = G;
    p.dist = dist;
    if (dist.kind != Dist::Block && tile <= 0) {
        // cyclic over single elements is meaningless for tile tasks: use 128-wide tasks
        tile = 128;
    }
    bool hetero = false;
    if (speeds && (int)speeds->size() == G && dist.kind == Dist::Block)
        for (double s : *speeds) hetero |= (s != (*speeds)[0]);
    // Worker grid for the overlapped exchange (runtime.exchange_overlapped): the B
    // column-panel all-gather is exposed, the A chunks stream in behind the
    // Worker's own chunk.  Choose Gr x Gc = G with Gc <= 4 (the own chunk is >= 1/4
    // of the Worker's work, enough to hide the other A chunks) minimising the
    // received B elements K*(N/Gc)*(1 - 1/Gr); ties -> fewer received elements in
    // total, then smaller Gr.  (G = 2: 1x2, 4: 1x4, 8: 2x4.)
    double best_b = std::numeric_limits<double>::infinity(), best_tot = best_b;
    for (int gr = 1; gr <= G; ++gr) {
        if (G % gr) continue;
        const int gc = G / gr;
        if (gc > 4 && gr < G) {
            bool alt = false;   // only skip if some grid with gc <= 4 exists
            for (int g2 = gr + 1; g2 <= G; ++g2)
                if (G % g2 == 0 && G / g2 <= 4) alt = true;
            if (alt) continue;
        }
        const double b = double(K) * (double(N) / gc) * (1.0 - 1.0 / gr);
        const double tot = (double(M) / gr) * double(K) * (1.0 - 1.0 / gc) + b;
        if (b < best_b * (1.0 - 1e-12) || (b <= best_b * (1.0 + 1e-12) && tot < best_tot * (1.0 - 1e-12))) {
            best_b = b;
            best_tot = tot;
            p.Gr = gr;
            p.Gc = gc;
        }
    }
    if (hetero) {
        p.Gr = G;
        p.Gc = 1;
    }
    if (tile > 0) {
        p.tile = tile;
        p.Tm = cdiv(M, tile);
        p.Tn = cdiv(N, tile);
    } else {
        // tile = 0: one task per Worker rectangle (continuous BLOCK split).
        p.tile = 0;
        p.Tm = p.Gr;
        p.Tn = p.Gc;
    }
    p.trow.resize(p.Gr + 1);
    p.tcol.resize(p.Gc + 1);
    p.row.resize(p.Gr + 1);
    p.col.resize(p.Gc + 1);
    if (hetero) {
        // task rows proportional to speed: boundary r = round(Tm * sum_{i<r} s_i / sum s)
        // (tile = 0: rows of C instead of task rows)
        double tot = 0;
        for (double s : *speeds) tot += s;
        const int64_t units = p.tile ? p.Tm : M;
        double acc = 0;
        for (int r = 0; r <= p.Gr; ++r) {
            const int64_t b = r == p.Gr ? units : (int64_t)std::llround(units * acc / tot);
            p.trow[r] = p.tile ? b : r;
            p.row[r] = p.tile ? std::min<int64_t>(b * p.tile, M) : b;
            if (r < p.Gr) acc += (*speeds)[r];
        }
    } else {
        for (int r = 0; r <= p.Gr; ++r) {
            p.trow[r] = (int64_t)r * p.Tm / p.Gr;  // floor(r*Tm/Gr): remainder to higher rows
            p.row[r] = p.tile ? std::min<int64_t>(p.trow[r] * p.tile, M) : (int64_t)r * M / p.Gr;
        }
    }
    for (int c = 0; c <= p.Gc; ++c) {
        p.tcol[c] = (int64_t)c * p.Tn / p.Gc;
        p.col[c] = p.tile ? std::min<int64_t>(p.tcol[c] * p.tile, N) : (int64_t)c * N / p.Gc;
    }
    return p;
}

// ---- hierarchical BLOCK (Hybrid PUs) ----
namespace {
struct TNode {
    int pu = -1;            // model PU index (Master / Hybrid), or the Worker's
    int worker = -1;        // group index for a leaf
    std::vector<int> kids;  // node indices, document order
    double weight = 0.0;    // total RELATIVE_SPEED of the subtree's group Workers
};

// Map C rows [r0, r1) (elements; task-row aligned) x all columns onto node n.
void place(const std::vector<TNode> &T, int n, int64_t r0, int64_t r1, int64_t M, int64_t N, int64_t K, int64_t tile,
           const std::vector<double> &speeds, int unit, Plan &P) {
    const TNode &nd = T[n];
    if (nd.worker >= 0) {
        P.wrect[nd.worker] = Rect{r0, r1, 0, N};
        P.wunit[nd.worker] = unit;
        return;
    }
    if (nd.kids.size() == 1) {
        place(T, nd.kids[0], r0, r1, M, N, K, tile, speeds, unit, P);
        return;
    }
    bool leaves = true;
    for (int k : nd.kids) leaves &= T[k].worker >= 0;
    if (leaves) {   // a PU controlling only Workers: the flat BLOCK plan on its band
        std::vector<double> sp;
        for (int k : nd.kids) sp.push_back(speeds[T[k].worker]);
        Plan sub = make_plan(r1 - r0, N, K, tile, (int)nd.kids.size(), DistSpec(), &sp);
        for (size_t i = 0; i < nd.kids.size(); ++i) {
            Rect R = sub.rect((int)i);
            R.row0 += r0;
            R.row1 += r0;
            P.wrect[T[nd.kids[i]].worker] = R;
            P.wunit[T[nd.kids[i]].worker] = unit;
        }
        return;
    }
    // row bands per child subtree, whole task rows, proportional to subtree speed
    const int64_t edge = tile > 0 ? tile : 1;
    const int64_t t0 = r0 / edge, units = (r1 - r0 + edge - 1) / edge;
    double tot = 0.0;
    for (int k : nd.kids) tot += T[k].weight;
    double acc = 0.0;
    int64_t prev = r0;
    for (size_t i = 0; i < nd.kids.size(); ++i) {
        acc += T[nd.kids[i]].weight;
        const int64_t tb = i + 1 == nd.kids.size() ? t0 + units : t0 + (int64_t)std::llround(units * acc / tot);
        const int64_t rb = std::min(r1, tb * edge);
        place(T, nd.kids[i], prev, std::max(prev, rb), M, N, K, tile, speeds, unit < 0 ? (int)i : unit, P);
        prev = std::max(prev, rb);
    }
}
}  // namespace

Plan make_plan_tree(int64_t M, int64_t N, int64_t K, int64_t tile, const Model &m, const std::vector<int> &gw,
                    DistSpec dist, const std::vector<double> &speeds) {
    const int G = (int)gw.size();
    Plan flat = make_plan(M, N, K, tile, G, dist, &speeds);
    if (dist.kind != Dist::Block || G < 2) return flat;
    // tree of the controlling PUs of the group's Workers
    std::vector<TNode> T(1);   // node 0: the virtual root above the Masters
    std::map<int, int> node_of;   // model PU -> node
    for (int w = 0; w < G; ++w) {
        std::vector<int> chain;   // Worker, its controllers ..., top-level PU
        for (int p = gw[w]; p >= 0; p = m.pus[p].parent) chain.push_back(p);
        int parent = 0;
        for (int i = (int)chain.size() - 1; i >= 0; --i) {
            auto it = node_of.find(chain[i]);
            int nd;
            if (it == node_of.end()) {
                nd = (int)T.size();
                T.push_back(TNode());
                T[nd].pu = chain[i];
                if (i == 0) T[nd].worker = w;
                node_of[chain[i]] = nd;
                T[parent].kids.push_back(nd);
            } else {
                nd = it->second;
            }
            T[nd].weight += speeds[w];
            parent = nd;
        }
        T[0].weight += speeds[w];
    }
    // flat when no PU below the Masters splits the group (all Workers are children of
    // one controller, possibly through a chain of single-child Hybrids)
    int n = 0;
    while (T[n].worker < 0 && T[n].kids.size() == 1) n = T[n].kids[0];
    bool leaves = T[n].worker < 0;
    for (int k : T[n].kids) leaves &= T[k].worker >= 0;
    if (leaves) return flat;
    Plan P = flat;
    P.wrect.assign(G, Rect());
    P.wunit.assign(G, -1);
    place(T, n, 0, M, M, N, K, tile, speeds, -1, P);
    return P;
}

std::string Plan::to_json(const std::vector<int> &workers, const std::vector<std::string> &ids) const {
    std::ostringstream o;
    o << "{\"M\":" << M << ",\"N\":" << N << ",\"K\":" << K << ",\"tile\":" << tile << ",\"G\":" << G
      << ",\"Gr\":" << Gr << ",\"Gc\":" << Gc << ",\"Tm\":" << Tm << ",\"Tn\":" << Tn
      << ",\"qb\":" << qb() << ",\"exchanged_elems\":" << (int64_t)exchanged_elems() << ",\"dist\":\""
      << (dist.kind == Dist::Block ? "BLOCK" : dist.kind == Dist::Cyclic ? "CYCLIC"
          : dist.kind == Dist::Dynamic ? "DYNAMIC" : "BLOCK-CYCLIC") << "\",\"dist_b\":"
      << dist.b << ",\"hierarchical\":" << (hierarchical() ? "true" : "false") << ",\"workers\":[";
    for (int w = 0; w < G; ++w) {
        Rect R = rect(w);
        int r = w / Gc, c = w % Gc;
        if (w) o << ",";
        if (hierarchical()) {   // explicit rectangle inside its Hybrid subtree's band
            const int64_t e = tile > 0 ? tile : 1;
            o << "{\"w\":" << w << ",\"id\":\"" << (w < (int)ids.size() ? json_escape(ids[w]) : "")
              << "\",\"unit\":" << wunit[w] << ",\"rows\":[" << R.row0 << "," << R.row1 << "],\"cols\":[" << R.col0
              << "," << R.col1 << "],\"task_rows\":[" << R.row0 / e << "," << (R.row1 + e - 1) / e
              << "],\"task_cols\":[" << R.col0 / e << "," << (R.col1 + e - 1) / e << "]}";
            continue;
        }
        if (dist.kind == Dist::Dynamic) {   // no static rectangle: tiles are claimed at run time
            o << "{\"w\":" << w << ",\"id\":\"" << (w < (int)ids.size() ? json_escape(ids[w]) : "")
              << "\",\"rows\":[0," << M << "],\"cols\":[0," << N << "],\"dynamic\":true}";
            continue;
        }
        o << "{\"w\":" << w << ",\"id\":\"" << (w < (int)ids.size() ? json_escape(ids[w]) : "") << "\""
          << ",\"r\":" << r << ",\"c\":" << c << ",\"rows\":[" << R.row0 << "," << R.row1 << "],\"cols\":["
          << R.col0 << "," << R.col1 << "],\"task_rows\":[" << trow[r] << "," << trow[r + 1]
          << "],\"task_cols\":[" << tcol[c] << "," << tcol[c + 1] << "],\"qa\":" << qa(w);
        if (dist.kind != Dist::Block) {
            o << ",\"row_segs\":[";
            auto rs = row_segs(r), cs = col_segs(c);
            for (size_t i = 0; i < rs.size(); ++i) o << (i ? "," : "") << "[" << rs[i].lo << "," << rs[i].hi << "]";
            o << "],\"col_segs\":[";
            for (size_t i = 0; i < cs.size(); ++i) o << (i ? "," : "") << "[" << cs[i].lo << "," << cs[i].hi << "]";
            o << "]";
        }
        o << "}";
    }
    (void)workers;
    o << "]}";
    return o.str();
}

}  // namespace pdl
