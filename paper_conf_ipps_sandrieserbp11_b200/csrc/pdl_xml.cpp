// pdl_xml.cpp -- see pdl_xml.hpp.
#include "pdl_xml.hpp"

#include <cctype>
#include <cstdlib>
#include <cstring>

namespace pdl {

std::string local_name(const std::string &q) {
    size_t p = q.find(':');
    return p == std::string::npos ? q : q.substr(p + 1);
}

std::string trim(const std::string &s) {
    size_t b = 0, e = s.size();
    while (b < e && std::isspace((unsigned char)s[b])) ++b;
    while (e > b && std::isspace((unsigned char)s[e - 1])) --e;
    return s.substr(b, e - b);
}

std::string XmlNode::local() const { return local_name(name); }

const std::string *XmlNode::attr(const char *ln) const {
    for (auto &kv : attrs)
        if (local_name(kv.first) == ln) return &kv.second;
    return nullptr;
}

namespace {

struct Parser {
    const std::string &s;
    size_t i = 0;
    int line = 1;
    explicit Parser(const std::string &d) : s(d) {}

    [[noreturn]] void fail(const std::string &m) { throw XmlError{m, line}; }
    bool eof() const { return i >= s.size(); }
    char peek(size_t k = 0) const { return i + k < s.size() ? s[i + k] : '\0'; }
    bool starts(const char *p) const { return s.compare(i, std::strlen(p), p) == 0; }
    void adv(size_t n = 1) {
        for (size_t k = 0; k < n && i < s.size(); ++k, ++i)
            if (s[i] == '\n') ++line;
    }
    void skip_ws() { while (!eof() && std::isspace((unsigned char)peek())) adv(); }

    void skip_until(const char *end, const char *what) {
        size_t p = s.find(end, i);
        if (p == std::string::npos) fail(std::string("unterminated ") + what);
        adv(p + std::strlen(end) - i);
    }

    // Misc: comments, processing instructions, doctype.
    bool skip_misc() {
        if (starts("<!--")) { skip_until("-->", "comment"); return true; }
        if (starts("<?")) { skip_until("?>", "processing instruction"); return true; }
        if (starts("<!DOCTYPE")) {
            int depth = 0;
            while (!eof()) {
                char c = peek();
                if (c == '[') ++depth;
                else if (c == ']') --depth;
                else if (c == '>' && depth <= 0) { adv(); return true; }
                adv();
            }
            fail("unterminated DOCTYPE");
        }
        return false;
    }

    static bool name_start(char c) {
        return std::isalpha((unsigned char)c) || c == '_' || c == ':' || (unsigned char)c >= 0x80;
    }
    static bool name_char(char c) {
        return name_start(c) || std::isdigit((unsigned char)c) || c == '-' || c == '.';
    }
    std::string name() {
        if (!name_start(peek())) fail("expected a name");
        size_t b = i;
        while (!eof() && name_char(peek())) adv();
        return s.substr(b, i - b);
    }

    static void put_utf8(std::string &o, unsigned long cp) {
        if (cp < 0x80) o += char(cp);
        else if (cp < 0x800) { o += char(0xC0 | (cp >> 6)); o += char(0x80 | (cp & 0x3F)); }
        else if (cp < 0x10000) {
            o += char(0xE0 | (cp >> 12)); o += char(0x80 | ((cp >> 6) & 0x3F));
            o += char(0x80 | (cp & 0x3F));
        } else {
            o += char(0xF0 | (cp >> 18)); o += char(0x80 | ((cp >> 12) & 0x3F));
            o += char(0x80 | ((cp >> 6) & 0x3F)); o += char(0x80 | (cp & 0x3F));
        }
    }

    // Decode one entity at s[i] == '&'.
    void entity(std::string &o) {
        size_t semi = s.find(';', i);
        if (semi == std::string::npos || semi - i > 12) fail("bad entity reference");
        std::string e = s.substr(i + 1, semi - i - 1);
        if (e == "lt") o += '<';
        else if (e == "gt") o += '>';
        else if (e == "amp") o += '&';
        else if (e == "quot") o += '"';
        else if (e == "apos") o += '\'';
        else if (!e.empty() && e[0] == '#') {
            char *endp = nullptr;
            unsigned long cp = (e.size() > 1 && (e[1] == 'x' || e[1] == 'X'))
                                   ? std::strtoul(e.c_str() + 2, &endp, 16)
                                   : std::strtoul(e.c_str() + 1, &endp, 10);
            if (!endp || *endp || cp == 0 || cp > 0x10FFFF) fail("bad character reference &" + e + ";");
            put_utf8(o, cp);
        } else {
            fail("unknown entity &" + e + ";");
        }
        adv(semi + 1 - i);
    }

    std::string attr_value() {
        char q = peek();
        if (q != '"' && q != '\'') fail("attribute value must be quoted");
        adv();
        std::string v;
        while (!eof() && peek() != q) {
            if (peek() == '<') fail("'<' in attribute value");
            if (peek() == '&') entity(v);
            else { v += peek(); adv(); }
        }
        if (eof()) fail("unterminated attribute value");
        adv();
        return v;
    }

    int depth = 0;
    static constexpr int kMaxDepth = 1024;   // recursion bound (descriptors are shallow trees)

    std::unique_ptr<XmlNode> element() {
        if (peek() != '<') fail("expected '<'");
        if (++depth > kMaxDepth) fail("element nesting deeper than 1024");
        struct DepthGuard {
            int &d;
            ~DepthGuard() { --d; }
        } guard{depth};
        auto n = std::make_unique<XmlNode>();
        n->line = line;
        adv();
        n->name = name();
        for (;;) {
            bool ws = std::isspace((unsigned char)peek());
            skip_ws();
            if (eof()) fail("unterminated start tag <" + n->name + ">");
            if (starts("/>")) { adv(2); return n; }
            if (peek() == '>') { adv(); break; }
            if (!ws) fail("expected whitespace before attribute in <" + n->name + ">");
            std::string an = name();
            skip_ws();
            if (peek() != '=') fail("expected '=' after attribute " + an);
            adv();
            skip_ws();
            std::string av = attr_value();
            for (auto &kv : n->attrs)
                if (kv.first == an) fail("duplicate attribute " + an);
            n->attrs.emplace_back(an, av);
        }
        // content
        for (;;) {
            if (eof()) fail("unterminated element <" + n->name + ">");
            if (starts("</")) {
                adv(2);
                std::string en = name();
                if (en != n->name) fail("mismatched end tag </" + en + "> for <" + n->name + ">");
                skip_ws();
                if (peek() != '>') fail("expected '>'");
                adv();
                return n;
            }
            if (starts("<![CDATA[")) {
                size_t p = s.find("]]>", i);
                if (p == std::string::npos) fail("unterminated CDATA");
                n->text += s.substr(i + 9, p - i - 9);
                adv(p + 3 - i);
                continue;
            }
            if (starts("<!--") || starts("<?")) { skip_misc(); continue; }
            if (peek() == '<') { n->children.push_back(element()); continue; }
            if (peek() == '&') { entity(n->text); continue; }
            n->text += peek();
            adv();
        }
    }

    std::unique_ptr<XmlNode> document() {
        // optional BOM
        if (s.size() >= 3 && (unsigned char)s[0] == 0xEF && (unsigned char)s[1] == 0xBB &&
            (unsigned char)s[2] == 0xBF)
            adv(3);
        for (;;) {
            skip_ws();
            if (!skip_misc()) break;
        }
        if (eof()) fail("empty document");
        auto root = element();
        for (;;) {
            skip_ws();
            if (eof()) break;
            if (!skip_misc()) fail("content after the root element");
        }
        return root;
    }
};

}  // namespace

std::unique_ptr<XmlNode> parse_xml(const std::string &doc) {
    Parser p(doc);
    return p.document();
}

}  // namespace pdl
