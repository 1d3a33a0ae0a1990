// host_sanitize.cpp -- the host-side PDL reader, machine model and mapper
// (csrc/pdl_xml.cpp, pdl_model.cpp, pdl_map.cpp) under AddressSanitizer +
// UndefinedBehaviorSanitizer (tests/test_host_sanitizers.py builds and runs it).
// Parses the golden descriptors and the shipped B200 descriptors, a seeded
// stream of mutated documents, and sweeps the mapper over shapes, Worker
// counts, tiles, distributions and speed weights, checking that every C
// element is owned exactly once.
#include <cstdio>
#include <cstdlib>
#include <fstream>
#include <random>
#include <sstream>
#include <string>
#include <vector>

#include "pdl_model.hpp"
#include "pdl_xml.hpp"

using namespace pdl;

static std::string slurp(const char *p) {
    std::ifstream f(p, std::ios::binary);
    std::stringstream ss;
    ss << f.rdbuf();
    return ss.str();
}

static int parse_ok(const std::string &doc) {
    try {
        auto root = parse_xml(doc);
        Model m = build_model(*root);
        (void)m.to_json();
        return 1;
    } catch (const XmlError &) {
        return 0;
    } catch (const ModelError &) {
        return 0;
    }
}

int main(int argc, char **argv) {
    std::vector<std::string> seeds;
    for (int i = 1; i < argc; ++i) seeds.push_back(slurp(argv[i]));
    int ok = 0, bad = 0;
    for (auto &s : seeds) {
        if (!parse_ok(s)) {
            fprintf(stderr, "seed failed to parse\n");
            return 2;
        }
    }
    std::mt19937_64 rng(42);
    const char *inserts[] = {"<", ">", "&", "\"", "'", "/", "=", "]]>", "<!--", "&#x0;", "<![CDATA[", "&#99999999;"};
    for (int n = 0; n < 20000; ++n) {
        std::string d = seeds[rng() % seeds.size()];
        int muts = 1 + rng() % 3;
        for (int k = 0; k < muts && !d.empty(); ++k) {
            size_t i = rng() % d.size();
            switch (rng() % 4) {
                case 0: d.resize(i); break;
                case 1: d[i] = (char)(rng() % 256); break;
                case 2: d.insert(i, inserts[rng() % (sizeof inserts / sizeof *inserts)]); break;
                default: d.erase(i, 1 + rng() % 30); break;
            }
        }
        (parse_ok(d) ? ok : bad)++;
    }
    // mapper sweep
    int plans = 0;
    for (int G = 1; G <= 8; ++G)
        for (int64_t M : {1, 7, 130, 1000})
            for (int64_t N : {1, 9, 257})
                for (int64_t tile : {0, 1, 16, 128})
                    for (int dk = 0; dk < 3; ++dk)
                        for (int hetero = 0; hetero < 2; ++hetero) {
                            DistSpec ds;
                            ds.kind = dk == 0 ? Dist::Block : dk == 1 ? Dist::Cyclic : Dist::BlockCyclic;
                            ds.b = dk == 2 ? 3 : 1;
                            std::vector<double> sp(G, 1.0);
                            if (hetero) sp[0] = 2.5;
                            Plan p = make_plan(M, N, 17, tile, G, ds, &sp);
                            std::vector<unsigned char> cover((size_t)(M * N), 0);
                            for (int w = 0; w < G; ++w)
                                for (const Seg &r : p.row_segs(w / p.Gc))
                                    for (const Seg &c : p.col_segs(w % p.Gc))
                                        for (int64_t i = r.lo; i < r.hi; ++i)
                                            for (int64_t j = c.lo; j < c.hi; ++j) cover[(size_t)(i * N + j)]++;
                            for (auto v : cover)
                                if (v != 1) {
                                    fprintf(stderr, "cover error G=%d M=%lld N=%lld tile=%lld dist=%d\n", G,
                                            (long long)M, (long long)N, (long long)tile, dk);
                                    return 3;
                                }
                            (void)p.to_json({}, {});
                            ++plans;
                        }
    printf("host_sanitize: %d mutated docs parsed, %d rejected, %d plans checked\n", ok, bad, plans);
    return 0;
}
