// pdl_xml.hpp -- minimal XML reader for PDL descriptors.
//
// PDL is "an XML-based platform description language" (PAPER.md SS III-B,
// L605-680).  The subset needed for descriptors: elements, attributes,
// comments, the <?xml?> header, <!DOCTYPE>, CDATA, the five predefined
// entities and numeric character references, and prefixed names
// (`ocl:name`, `xsi:type`, Listing 2).  No external dependency.
#pragma once
#include <memory>
#include <string>
#include <utility>
#include <vector>

namespace pdl {

struct XmlNode {
    std::string name;                                       // qualified name as written
    std::vector<std::pair<std::string, std::string>> attrs; // qualified name -> value
    std::vector<std::unique_ptr<XmlNode>> children;
    std::string text;                                       // concatenated character data
    int line = 0;

    std::string local() const;                              // name without prefix
    const std::string *attr(const char *local_name) const;  // match by local name
};

struct XmlError {
    std::string msg;
    int line;
};

// Parse a document; throws XmlError.  Returns the root element.
std::unique_ptr<XmlNode> parse_xml(const std::string &doc);

std::string local_name(const std::string &qname);
std::string trim(const std::string &s);

}  // namespace pdl
