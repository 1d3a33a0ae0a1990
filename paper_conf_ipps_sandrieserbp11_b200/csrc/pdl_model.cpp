// pdl_model.cpp -- PDL descriptor -> hierarchical machine model (see header).
#include "pdl_model.hpp"

#include <algorithm>
#include <cctype>
#include <cmath>
#include <cstdlib>
#include <set>
#include <functional>
#include <sstream>

namespace pdl {

const char *kind_name(PUKind k) {
    switch (k) {
        case PUKind::Master: return "Master";
        case PUKind::Hybrid: return "Hybrid";
        default: return "Worker";
    }
}

std::string lower(const std::string &s) {
    std::string o(s);
    for (auto &c : o) c = (char)std::tolower((unsigned char)c);
    return o;
}

std::string norm_key(const std::string &name) {
    std::string o;
    for (char c : trim(name)) {
        if (c == ' ' || c == '-' || c == '\t') {
            if (o.empty() || o.back() != '_') o += '_';
        } else {
            o += (char)std::toupper((unsigned char)c);
        }
    }
    return o;
}

std::string json_escape(const std::string &s) {
    std::string o;
    for (unsigned char c : s) {
        switch (c) {
            case '"': o += "\\\""; break;
            case '\\': o += "\\\\"; break;
            case '\n': o += "\\n"; break;
            case '\r': o += "\\r"; break;
            case '\t': o += "\\t"; break;
            default:
                if (c < 0x20) {
                    char b[8];
                    snprintf(b, sizeof b, "\\u%04x", c);
                    o += b;
                } else {
                    o += (char)c;
                }
        }
    }
    return o;
}

// R10: sizes with unit B / kB / MB / GB / TB are powers of 1024 (Listing 2's
// GLOBAL MEM SIZE 1572864 kB is the GTX 480's 1.5 GiB, L901).
bool value_bytes(const Property &p, uint64_t *out) {
    std::string u = lower(trim(p.unit));
    double mult;
    if (u == "b" || u == "byte" || u == "bytes") mult = 1.0;
    else if (u == "kb" || u == "kib") mult = 1024.0;
    else if (u == "mb" || u == "mib") mult = 1024.0 * 1024.0;
    else if (u == "gb" || u == "gib") mult = 1024.0 * 1024.0 * 1024.0;
    else if (u == "tb" || u == "tib") mult = 1024.0 * 1024.0 * 1024.0 * 1024.0;
    else return false;
    std::string v = trim(p.value);
    if (v.empty()) return false;
    char *end = nullptr;
    double x = std::strtod(v.c_str(), &end);
    if (!end || *end || !(x >= 0) || !std::isfinite(x)) return false;
    *out = (uint64_t)std::llround(x * mult);
    return true;
}

const Property *Model::prop(int pu, const std::string &key) const {
    std::string k = norm_key(key);
    for (auto &p : pus[pu].props)
        if (p.key == k) return &p;
    if (k == "ARCHITECTURE") return prop(pu, "ARCH");  // R9: ARCH (Fig. 1) alias
    return nullptr;
}

Property *Model::prop_mut(int pu, const std::string &key) {
    return const_cast<Property *>(prop(pu, key));
}

bool Model::is_gpu_worker(int pu) const {
    if (pus[pu].kind != PUKind::Worker) return false;
    const Property *a = prop(pu, "ARCHITECTURE");
    return a && lower(trim(a->value)) == "gpu";
}

bool Model::in_group(int pu, const std::string &g) const {
    for (int p = pu; p >= 0; p = pus[p].parent)
        for (auto &x : pus[p].groups)
            if (x == g) return true;
    return false;
}

std::vector<int> Model::all_gpu_workers() const {
    std::vector<int> v;
    for (int i = 0; i < (int)pus.size(); ++i)
        if (is_gpu_worker(i)) v.push_back(i);
    return v;
}

std::vector<int> Model::group_workers(const char *group) const {
    std::vector<int> v;
    for (int i = 0; i < (int)pus.size(); ++i)
        if (is_gpu_worker(i) && (!group || in_group(i, group))) v.push_back(i);
    return v;
}

// R8: an Interconnect names template ids; from == to on a replicated PU joins
// all pairs of its instances; interconnects are bidirectional.
bool Model::ic_between(int a, int b, const std::string &type_ci) const {
    const std::string &ta = pus[a].tid, &tb = pus[b].tid;
    for (auto &ic : ics) {
        if (!type_ci.empty() && lower(ic.type) != lower(type_ci)) continue;
        if ((ic.from == ta && ic.to == tb) || (ic.from == tb && ic.to == ta)) return true;
    }
    return false;
}

std::string Model::ic_type_between(int a, int b) const {
    const std::string &ta = pus[a].tid, &tb = pus[b].tid;
    for (auto &ic : ics)
        if ((ic.from == ta && ic.to == tb) || (ic.from == tb && ic.to == ta)) return ic.type;
    return "";
}

namespace {

bool is_pu(const XmlNode &n) {
    std::string l = n.local();
    return l == "Master" || l == "Hybrid" || l == "Worker";
}

PUKind pu_kind(const XmlNode &n) {
    std::string l = n.local();
    if (l == "Master") return PUKind::Master;
    if (l == "Hybrid") return PUKind::Hybrid;
    return PUKind::Worker;
}

[[noreturn]] void fail(const std::string &m, int line) { throw ModelError{m, line}; }

Property parse_property(const XmlNode &n) {
    Property p;
    if (auto f = n.attr("fixed")) {
        std::string v = lower(trim(*f));
        if (v == "true" || v == "1") p.fixed = true;
        else if (v == "false" || v == "0") p.fixed = false;
        else fail("Property attribute fixed must be true or false, got '" + *f + "'", n.line);
        p.fixed_given = true;
    }
    if (auto t = n.attr("type")) p.xsi_type = *t;
    bool has_name = false;
    for (auto &c : n.children) {
        std::string l = c->local();
        if (l == "name") { p.name = trim(c->text); has_name = true; }
        else if (l == "value") {
            p.value = trim(c->text);
            if (auto u = c->attr("unit")) p.unit = trim(*u);
        }
    }
    // also accept <Property name=".." value=".."/>
    if (!has_name) {
        if (auto a = n.attr("name")) { p.name = trim(*a); has_name = true; }
        if (auto a = n.attr("value")) p.value = trim(*a);
        if (auto a = n.attr("unit")) p.unit = trim(*a);
    }
    if (!has_name || p.name.empty()) fail("Property without a <name>", n.line);
    p.key = norm_key(p.name);
    return p;
}

void parse_descriptor(const XmlNode &d, std::vector<Property> &out) {
    for (auto &c : d.children)
        if (c->local() == "Property") out.push_back(parse_property(*c));
}

struct Template {
    const XmlNode *node;
    PUKind kind;
    std::string tid;
    int quantity;
    int parent_t;  // template index of the controlling PU, -1 at top level
};

int parse_quantity(const XmlNode &n) {
    const std::string *q = n.attr("quantity");
    if (!q) return 1;
    std::string v = trim(*q);
    if (v.empty()) fail("empty quantity on <" + n.name + ">", n.line);
    for (char c : v)
        if (!std::isdigit((unsigned char)c)) fail("quantity must be a positive integer, got '" + *q + "'", n.line);
    long x = std::strtol(v.c_str(), nullptr, 10);
    if (x < 1 || x > 65536) fail("quantity must be >= 1, got '" + *q + "'", n.line);
    return (int)x;
}

void collect(const XmlNode &n, int parent_t, std::vector<Template> &ts, std::vector<Interconnect> &ics,
             std::set<std::string> &ids) {
    PUKind k = pu_kind(n);
    // Structural rules of SS III-A.
    if (k == PUKind::Master && parent_t >= 0)
        fail("Master PU nested inside another PU: Masters are only defined on the highest "
             "hierarchical level (L495-503)", n.line);
    if (k != PUKind::Master && parent_t < 0)
        fail(std::string(kind_name(k)) + " PU at top level: Workers and Hybrids must be "
             "controlled by a Master or Hybrid PU (L505-531)", n.line);
    if (parent_t >= 0 && ts[parent_t].kind == PUKind::Worker)
        fail("PU nested inside a Worker: Workers are leaf nodes (L505-511)", n.line);
    const std::string *id = n.attr("id");
    if (!id || trim(*id).empty()) fail("<" + n.name + "> without an id", n.line);
    std::string tid = trim(*id);
    if (!ids.insert(tid).second) fail("duplicate PU id '" + tid + "'", n.line);
    int me = (int)ts.size();
    ts.push_back(Template{&n, k, tid, parse_quantity(n), parent_t});
    int nchild = 0;
    for (auto &c : n.children) {
        if (is_pu(*c)) {
            collect(*c, me, ts, ics, ids);
            ++nchild;
        } else if (c->local() == "Interconnect") {
            Interconnect ic;
            ic.line = c->line;
            if (auto a = c->attr("type")) ic.type = trim(*a);
            if (auto a = c->attr("from")) ic.from = trim(*a);
            if (auto a = c->attr("to")) ic.to = trim(*a);
            if (auto a = c->attr("scheme")) ic.scheme = trim(*a);
            for (auto &d : c->children)
                if (d->local() == "ICDescriptor") parse_descriptor(*d, ic.props);
            if (ic.from.empty() || ic.to.empty()) fail("Interconnect without from/to", c->line);
            ics.push_back(ic);
        }
    }
    if (k == PUKind::Hybrid && nchild == 0)
        fail("Hybrid PU '" + tid + "' without controlled PUs: Hybrids are inner nodes (L513-531)",
             n.line);
}

}  // namespace

Model build_model(const XmlNode &root) {
    std::vector<Template> ts;
    Model m;
    std::set<std::string> ids;
    if (is_pu(root)) {
        collect(root, -1, ts, m.ics, ids);
    } else {
        // wrapper root (e.g. <Platform>) holding co-existing Masters (L495-503)
        for (auto &c : root.children) {
            if (is_pu(*c)) collect(*c, -1, ts, m.ics, ids);
            else if (c->local() == "Interconnect") {
                Interconnect ic;
                ic.line = c->line;
                if (auto a = c->attr("type")) ic.type = trim(*a);
                if (auto a = c->attr("from")) ic.from = trim(*a);
                if (auto a = c->attr("to")) ic.to = trim(*a);
                if (auto a = c->attr("scheme")) ic.scheme = trim(*a);
                for (auto &d : c->children)
                    if (d->local() == "ICDescriptor") parse_descriptor(*d, ic.props);
                if (ic.from.empty() || ic.to.empty()) fail("Interconnect without from/to", c->line);
                m.ics.push_back(ic);
            }
        }
    }
    bool any_master = false;
    for (auto &t : ts) any_master |= (t.kind == PUKind::Master);
    if (!any_master) fail("descriptor has no Master PU (a Master marks the starting point of execution, L495-503)",
                          root.line);
    for (auto &ic : m.ics) {
        if (!ids.count(ic.from)) fail("Interconnect from unknown PU id '" + ic.from + "'", ic.line);
        if (!ids.count(ic.to)) fail("Interconnect to unknown PU id '" + ic.to + "'", ic.line);
    }

    // Total instance count per template (replication multiplies down the tree).
    std::vector<int64_t> total(ts.size());
    for (size_t t = 0; t < ts.size(); ++t) {
        int64_t mult = ts[t].quantity;
        if (ts[t].parent_t >= 0) mult *= total[ts[t].parent_t];
        if (mult > 65536) fail("quantity expansion too large", ts[t].node->line);
        total[t] = mult;
    }
    std::vector<int> counter(ts.size(), 0);

    // Expand instances in pre-order (R7: quantity q -> q identical PUs).
    std::function<void(int, int)> expand = [&](int t, int parent_inst) {
        const Template &T = ts[t];
        for (int j = 0; j < T.quantity; ++j) {
            PU pu;
            pu.kind = T.kind;
            pu.tid = T.tid;
            pu.quantity = T.quantity;
            pu.replica = counter[t]++;
            pu.id = total[t] == 1 ? T.tid : T.tid + "." + std::to_string(pu.replica);
            pu.parent = parent_inst;
            pu.line = T.node->line;
            for (auto &c : T.node->children) {
                std::string l = c->local();
                if (l == "PUDescriptor") parse_descriptor(*c, pu.props);
                else if (l == "MemoryRegion") {
                    MemoryRegion mr;
                    if (auto a = c->attr("id")) mr.id = trim(*a);
                    for (auto &d : c->children) {
                        if (d->local() == "MRDescriptor") parse_descriptor(*d, mr.props);
                        else if (d->local() == "Property") mr.props.push_back(parse_property(*d));
                    }
                    pu.mrs.push_back(mr);
                } else if (l == "LogicGroupAttribute") {
                    std::string g = trim(c->text);
                    if (g.empty())
                        if (auto a = c->attr("name")) g = trim(*a);
                    if (g.empty())
                        if (auto a = c->attr("value")) g = trim(*a);
                    if (!g.empty()) pu.groups.push_back(g);
                }
            }
            int me = (int)m.pus.size();
            m.pus.push_back(pu);
            if (parent_inst >= 0) m.pus[parent_inst].children.push_back(me);
            else m.masters.push_back(me);
            for (size_t c = 0; c < ts.size(); ++c)
                if (ts[c].parent_t == t) expand((int)c, me);
        }
    };
    for (size_t t = 0; t < ts.size(); ++t)
        if (ts[t].parent_t < 0) expand((int)t, -1);
    return m;
}

static void props_json(std::ostringstream &o, const std::vector<Property> &ps) {
    o << "{";
    for (size_t i = 0; i < ps.size(); ++i) {
        auto &p = ps[i];
        if (i) o << ",";
        o << "\"" << json_escape(p.key) << "\":{\"name\":\"" << json_escape(p.name) << "\",\"value\":\""
          << json_escape(p.value) << "\",\"unit\":\"" << json_escape(p.unit) << "\",\"fixed\":"
          << (p.fixed ? "true" : "false");
        if (!p.xsi_type.empty()) o << ",\"xsi_type\":\"" << json_escape(p.xsi_type) << "\"";
        uint64_t b;
        if (value_bytes(p, &b)) o << ",\"bytes\":" << b;
        o << "}";
    }
    o << "}";
}

std::string Model::ics_json() const {
    std::ostringstream o;
    o << "[";
    for (size_t i = 0; i < ics.size(); ++i) {
        auto &ic = ics[i];
        if (i) o << ",";
        o << "{\"type\":\"" << json_escape(ic.type) << "\",\"from\":\"" << json_escape(ic.from)
          << "\",\"to\":\"" << json_escape(ic.to) << "\",\"scheme\":\"" << json_escape(ic.scheme)
          << "\",\"props\":";
        props_json(o, ic.props);
        o << "}";
    }
    o << "]";
    return o.str();
}

std::string Model::to_json() const {
    std::ostringstream o;
    o << "{\"pus\":[";
    for (size_t i = 0; i < pus.size(); ++i) {
        auto &p = pus[i];
        if (i) o << ",";
        o << "{\"id\":\"" << json_escape(p.id) << "\",\"tid\":\"" << json_escape(p.tid) << "\",\"kind\":\""
          << kind_name(p.kind) << "\",\"quantity\":" << p.quantity << ",\"parent\":";
        if (p.parent >= 0) o << "\"" << json_escape(pus[p.parent].id) << "\"";
        else o << "null";
        o << ",\"children\":[";
        for (size_t c = 0; c < p.children.size(); ++c)
            o << (c ? "," : "") << "\"" << json_escape(pus[p.children[c]].id) << "\"";
        o << "],\"groups\":[";
        for (size_t g = 0; g < p.groups.size(); ++g) o << (g ? "," : "") << "\"" << json_escape(p.groups[g]) << "\"";
        o << "],\"gpu\":" << (is_gpu_worker((int)i) ? "true" : "false") << ",\"device\":" << p.device
          << ",\"props\":";
        props_json(o, p.props);
        o << ",\"mrs\":[";
        for (size_t r = 0; r < p.mrs.size(); ++r) {
            if (r) o << ",";
            o << "{\"id\":\"" << json_escape(p.mrs[r].id) << "\",\"props\":";
            props_json(o, p.mrs[r].props);
            o << "}";
        }
        o << "]}";
    }
    o << "],\"masters\":[";
    for (size_t i = 0; i < masters.size(); ++i) o << (i ? "," : "") << "\"" << json_escape(pus[masters[i]].id) << "\"";
    o << "],\"interconnects\":" << ics_json() << "}";
    return o.str();
}

}  // namespace pdl
