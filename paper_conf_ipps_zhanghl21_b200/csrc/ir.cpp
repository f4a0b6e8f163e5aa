// IR text -> adjacency-list graph (Fig. 10: "iterate the IR ... obtain the
// inputs/outputs of each operator to build a graph with adjacency-lists").  Grammar: include/duet.h.
#include <algorithm>
#include <cctype>
#include <cstring>
#include <queue>

#include "common.h"

namespace duet {

Graph::~Graph() = default;

const char* dtype_name(int d) {
  switch (d) {
    case kF32: return "f32";
    case kBF16: return "bf16";
    case kI32: return "i32";
    case kI64: return "i64";
  }
  return "?";
}

int64_t Node::attr_int(const std::string& k, int64_t dflt) const {
  auto it = attrs.find(k);
  if (it == attrs.end()) return dflt;
  char* end = nullptr;
  long long v = strtoll(it->second.c_str(), &end, 10);
  if (!end || *end) fail(DUET_EPARSE, "attribute " + k + " of %" + name + " is not an integer");
  return v;
}

std::string Node::attr_str(const std::string& k, const std::string& dflt) const {
  auto it = attrs.find(k);
  return it == attrs.end() ? dflt : it->second;
}

namespace {

struct Lexer {
  const std::string& s;
  size_t i = 0;
  int line;
  explicit Lexer(const std::string& str, int ln) : s(str), line(ln) {}
  [[noreturn]] void err(const std::string& m) {
    fail(DUET_EPARSE, "IR line " + std::to_string(line) + ": " + m + ": '" + s + "'");
  }
  void ws() {
    while (i < s.size() && isspace((unsigned char)s[i])) ++i;
  }
  bool eof() {
    ws();
    return i >= s.size();
  }
  bool peek(char c) {
    ws();
    return i < s.size() && s[i] == c;
  }
  void expect(char c) {
    ws();
    if (i >= s.size() || s[i] != c) err(std::string("expected '") + c + "'");
    ++i;
  }
  std::string ident() {  // [A-Za-z_][\w.]*  (also digits-leading for attr values)
    ws();
    size_t b = i;
    while (i < s.size() && (isalnum((unsigned char)s[i]) || s[i] == '_' || s[i] == '.' || s[i] == '-' ||
                            s[i] == '+'))
      ++i;
    if (b == i) err("expected a name");
    return s.substr(b, i - b);
  }
  std::string word() {
    ws();
    size_t b = i;
    while (i < s.size() && (isalnum((unsigned char)s[i]) || s[i] == '_')) ++i;
    return s.substr(b, i - b);
  }
};

int parse_dtype(Lexer& L) {
  std::string d = L.word();
  if (d == "f32") return kF32;
  if (d == "bf16") return kBF16;
  if (d == "i32") return kI32;
  if (d == "i64") return kI64;
  L.err("unknown dtype '" + d + "'");
}

std::vector<int64_t> parse_shape(Lexer& L) {
  std::vector<int64_t> sh;
  L.expect('[');
  L.ws();
  if (L.peek(']')) {
    L.expect(']');
    return sh;
  }
  while (true) {
    std::string w = L.word();
    if (w.empty()) L.err("expected a dimension");
    for (char c : w)
      if (!isdigit((unsigned char)c)) L.err("bad dimension '" + w + "'");
    sh.push_back(std::stoll(w));
    if (L.peek(',')) {
      L.expect(',');
      continue;
    }
    L.expect(']');
    break;
  }
  if (sh.size() > DUET_MAX_DIMS) L.err("too many dimensions");
  return sh;
}

}  // namespace

Graph* parse_ir(const char* text, size_t len) {
  std::unique_ptr<Graph> g(new Graph());
  std::string all(text, len);
  std::vector<std::string> out_names;
  size_t pos = 0;
  int ln = 0;
  while (pos <= all.size()) {
    size_t e = all.find('\n', pos);
    if (e == std::string::npos) e = all.size();
    std::string line = all.substr(pos, e - pos);
    pos = e + 1;
    ++ln;
    size_t h = line.find('#');
    if (h != std::string::npos) line = line.substr(0, h);
    Lexer L(line, ln);
    if (L.eof()) {
      if (e == all.size()) break;
      continue;
    }
    if (L.peek('%')) {
      L.expect('%');
      Node n;
      n.name = L.ident();
      L.expect('=');
      n.op = L.word();
      if (n.op.empty()) L.err("expected an operator");
      L.expect('(');
      if (!L.peek(')')) {
        while (true) {
          L.ws();
          if (!(L.peek('%') || L.peek('@'))) L.err("argument must start with % or @");
          char k = L.s[L.i++];
          n.args.push_back({k, L.ident()});
          if (L.peek(',')) {
            L.expect(',');
            continue;
          }
          break;
        }
      }
      L.expect(')');
      if (L.peek('{')) {
        L.expect('{');
        if (!L.peek('}')) {
          while (true) {
            std::string k = L.word();
            if (k.empty()) L.err("expected an attribute name");
            L.expect('=');
            n.attrs[k] = L.ident();
            if (L.peek(',')) {
              L.expect(',');
              continue;
            }
            break;
          }
        }
        L.expect('}');
      }
      L.expect(':');
      n.dtype = parse_dtype(L);
      n.shape = parse_shape(L);
      if (!L.eof()) L.err("trailing characters");
      if (g->by_name.count(n.name)) L.err("duplicate value %" + n.name);
      n.id = (int)g->nodes.size();
      g->by_name[n.name] = n.id;
      g->nodes.push_back(std::move(n));
      if (e == all.size()) break;
      continue;
    }
    std::string kw = L.word();
    if (kw == "param") {
      L.expect('@');
      std::string name = L.ident();
      L.expect(':');
      ParamDecl d;
      d.dtype = parse_dtype(L);
      d.shape = parse_shape(L);
      if (!L.eof()) L.err("trailing characters");
      if (g->params.count(name)) L.err("duplicate parameter @" + name);
      g->params[name] = d;
      g->param_order.push_back(name);
    } else if (kw == "output") {
      while (true) {
        L.expect('%');
        out_names.push_back(L.ident());
        if (L.peek(',')) {
          L.expect(',');
          continue;
        }
        break;
      }
      if (!L.eof()) L.err("trailing characters");
    } else {
      L.err("cannot parse");
    }
    if (e == all.size()) break;
  }
  // resolve names
  for (auto& n : g->nodes) {
    std::set<int> ins;
    for (auto& a : n.args) {
      if (a.first == '%') {
        auto it = g->by_name.find(a.second);
        if (it == g->by_name.end()) fail(DUET_EPARSE, "undefined value %" + a.second);
        ins.insert(it->second);
        n.arg_nodes.push_back(it->second);
      } else {
        if (!g->params.count(a.second)) fail(DUET_EPARSE, "undefined parameter @" + a.second);
        n.params.push_back(a.second);
      }
    }
    n.inputs.assign(ins.begin(), ins.end());
    if (n.op == "input") g->input_nodes.push_back(n.id);
  }
  std::set<int> outs;
  for (auto& nm : out_names) {
    auto it = g->by_name.find(nm);
    if (it == g->by_name.end()) fail(DUET_EPARSE, "undefined output %" + nm);
    if (!outs.count(it->second)) g->outputs.push_back(it->second);
    outs.insert(it->second);
  }
  std::sort(g->outputs.begin(), g->outputs.end());
  // Kahn, smallest ready id first
  int n = (int)g->nodes.size();
  std::vector<int> indeg(n);
  std::vector<std::vector<int>> cons(n);
  for (auto& nd : g->nodes) {
    indeg[nd.id] = (int)nd.inputs.size();
    for (int u : nd.inputs) cons[u].push_back(nd.id);
  }
  std::priority_queue<int, std::vector<int>, std::greater<int>> ready;
  for (int i = 0; i < n; ++i)
    if (!indeg[i]) ready.push(i);
  while (!ready.empty()) {
    int u = ready.top();
    ready.pop();
    g->topo.push_back(u);
    for (int v : cons[u])
      if (--indeg[v] == 0) ready.push(v);
  }
  if ((int)g->topo.size() != n) fail(DUET_ECYCLE, "IR graph has a cycle");
  return g.release();
}

}  // namespace duet
