// pdl_model.hpp -- the hierarchical machine model built from a PDL descriptor.
//
// PAPER.md SS III-A (L472-603): processing units of three classes --
//   Master  "feature rich, general-purpose ... starting point for execution
//            of a program ... only defined on the highest hierarchical level
//            but may co-exist with other Masters" (L495-503);
//   Worker  "specialized compute resource ... leaf nodes ... must be
//            controlled by Master or Hybrid PUs" (L505-511);
//   Hybrid  "act as Master and Worker ... inner nodes ... must always be
//            controlled either by other Hybrid or Master units" (L513-531);
// plus MemoryRegions (L577-589) and Interconnects (L591-603).  SS III-B lists
// the XML entity set (L668-680) and the extensible Descriptor/Property pair
// (L682-708); fixed / unfixed properties (L737-747); LogicGroupAttribute
// group identifiers (L735-737).
#pragma once
#include <cstdint>
#include <map>
#include <string>
#include <vector>

#include "pdl_xml.hpp"

namespace pdl {

enum class PUKind { Master, Hybrid, Worker };
const char *kind_name(PUKind k);

struct Property {
    std::string name;       // as written (local name content of <name>)
    std::string key;        // normalised: upper case, ' ' and '-' -> '_'
    std::string value;
    std::string unit;       // <value unit="kB">
    std::string xsi_type;   // Property xsi:type (L876-886), kept as metadata
    bool fixed = true;      // fixed="false" -> editable by tools/runtime (L737-747)
    bool fixed_given = false;
};

struct MemoryRegion {
    std::string id;
    std::vector<Property> props;
};

struct Interconnect {
    std::string type, from, to, scheme;   // L827: type="rDMA" from="0" to="1" scheme=""
    std::vector<Property> props;          // ICDescriptor
    int line = 0;
};

struct PU {
    PUKind kind = PUKind::Worker;
    std::string tid;            // template id as written (id="1")
    std::string id;             // instance id: tid, or tid.j for quantity > 1 (R7)
    int replica = 0;            // j
    int quantity = 1;           // of the template
    int parent = -1;            // controlling PU instance (index), -1 at top level
    std::vector<int> children;
    std::vector<Property> props;            // PUDescriptor
    std::vector<MemoryRegion> mrs;
    std::vector<std::string> groups;        // LogicGroupAttribute values (own)
    int line = 0;
    // device binding (gpu Workers)
    int device = -1;
};

struct Model {
    std::vector<PU> pus;                    // instances, document order (pre-order)
    std::vector<Interconnect> ics;          // as written (template ids)
    std::vector<int> masters;

    const Property *prop(int pu, const std::string &key) const;
    Property *prop_mut(int pu, const std::string &key);
    bool is_gpu_worker(int pu) const;       // Worker with ARCHITECTURE/ARCH == gpu (R9)
    bool in_group(int pu, const std::string &group) const;  // own or ancestor LogicGroupAttribute
    std::vector<int> group_workers(const char *group) const;  // gpu Workers, document order
    std::vector<int> all_gpu_workers() const;
    bool ic_between(int a, int b, const std::string &type_ci) const;
    // type of the first Interconnect joining PU instances a and b ("" if none)
    std::string ic_type_between(int a, int b) const;
    std::string to_json() const;
    std::string ics_json() const;
};

struct ModelError {
    std::string msg;
    int line;
};

// Build + validate + expand quantities.  Throws ModelError / XmlError.
Model build_model(const XmlNode &root);

std::string norm_key(const std::string &name);
// Parse "<value unit=...>" into bytes when it is a size (R10: kB = 1024 B).
bool value_bytes(const Property &p, uint64_t *out);
std::string json_escape(const std::string &s);
std::string lower(const std::string &s);

// ---- mapping (pdl_map.cpp) ----
struct Rect {
    int64_t row0 = 0, row1 = 0, col0 = 0, col1 = 0;
};

// Data distributions of the execute annotation (L1200-1206: "block, cyclic,
// block-cyclic ... and optional sizes").
// DYNAMIC (the paper's future-work dynamic scheduler, L1556-1562):
// no static assignment -- the Workers' kernels claim tiles from a shared counter.
enum class Dist { Block, Cyclic, BlockCyclic, Dynamic };
struct DistSpec {
    Dist kind = Dist::Block;
    int64_t b = 1;   // tasks per cyclic block (CYCLIC = BLOCK-CYCLIC:1)
};
// Parse "BLOCK", "CYCLIC", "BLOCK-CYCLIC[:b]", "DYNAMIC" (case-insensitive; NULL = BLOCK).
// Returns false for an unknown name or a bad size.
bool parse_dist(const char *s, DistSpec *out);

struct Seg {
    int64_t lo = 0, hi = 0;   // element range [lo, hi)
};

struct Plan {
    int64_t M = 0, N = 0, K = 0, tile = 0;   // tile: effective task edge (0 = per-Worker blocks)
    int G = 0, Gr = 0, Gc = 0;
    DistSpec dist;
    int64_t Tm = 0, Tn = 0;                  // task grid
    std::vector<int64_t> trow, tcol;         // BLOCK: task-row / task-col boundaries per grid row / col
    std::vector<int64_t> row, col;           // BLOCK: element boundaries (Gr+1, Gc+1)
    // Hierarchical BLOCK through Hybrid PUs: explicit per-Worker rectangles and the
    // index of the Master's child subtree (level-1 unit) holding each Worker; empty
    // for a flat plan
    std::vector<Rect> wrect;
    std::vector<int> wunit;
    bool hierarchical() const { return !wrect.empty(); }
    Rect rect(int w) const;                  // BLOCK: the Worker's rectangle, w = r*Gc + c
    int64_t qa(int w) const;                 // rows per A chunk for Worker w
    int64_t qb() const;                      // K-rows per B chunk
    double exchanged_elems() const;          // received by all Workers (A + B)
    // any distribution: the Worker's C row / column segments (merged when adjacent)
    std::vector<Seg> row_segs(int r) const;
    std::vector<Seg> col_segs(int c) const;
    std::string to_json(const std::vector<int> &workers, const std::vector<std::string> &ids) const;
};

// Choose Gr x Gc = G (Gc <= 4) minimising the exposed exchange, the received B
// elements K*(N/Gc)*(1 - 1/Gr) (the A chunks overlap the kernels); ties -> fewer
// received elements in total, then smaller Gr.  BLOCK distributes task rows / cols (L1200-1206): grid row
// r gets task rows [floor(r*Tm/Gr), floor((r+1)*Tm/Gr)); CYCLIC / BLOCK-CYCLIC:b
// give grid row r the b-task blocks q with q % Gr == r (columns likewise).
//
// Heterogeneous Workers (the paper's GTX480 + GTX285 box,
// L1398-1402): when `speeds` (PDL property RELATIVE_SPEED of each Worker) are
// not all equal, BLOCK becomes a 1-D row split (Gr = G, Gc = 1) with task rows
// proportional to speed (cumulative rounding), so every Worker finishes together.
Plan make_plan(int64_t M, int64_t N, int64_t K, int64_t tile, int G, DistSpec dist = DistSpec(),
               const std::vector<double> *speeds = nullptr);

// Mapping through the PU hierarchy (Hybrid PUs "act as Master and
// Worker ... inner nodes", L513-531): the group's Workers are arranged in the tree
// of their controlling PUs below the Master.  Where a PU controls more than one
// subtree holding group Workers, BLOCK splits its C block into row bands, one per
// subtree in document order, sized by the subtree's total RELATIVE_SPEED in whole
// task rows (cumulative rounding); a PU whose children are all Workers maps its
// band with make_plan.  A flat tree (every Worker directly under the Master, or a
// single chain) gives exactly make_plan.  gw = the group's Workers (PU indices,
// document order); dist other than BLOCK ignores the hierarchy.
Plan make_plan_tree(int64_t M, int64_t N, int64_t K, int64_t tile, const Model &m, const std::vector<int> &gw,
                    DistSpec dist, const std::vector<double> &speeds);

// RELATIVE_SPEED of the group's Workers (1 when absent or invalid).
std::vector<double> worker_speeds(const Model &m, const std::vector<int> &workers);

}  // namespace pdl
