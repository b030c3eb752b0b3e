// Update-tree exploration (§4.5) as explicit state machines.  Semantics are
// step-for-step those of the plain model in oracle/tuner.py (checked by tests/test_tuner_native.py
// on identical trees and cost tables: same trial sequence, same final configuration).
#include "tuner.h"

#include <cctype>
#include <cmath>
#include <limits>
#include <sstream>
#include <stdexcept>

namespace astra {
namespace tuner {

std::string ProfileIndex::key(int ctx, const std::string& node, const std::string& choice, int bucket, int se) {
  std::ostringstream o;
  o << "ctx=" << ctx << "|b=" << bucket << "|se=" << se << "|node=" << node << "|choice=" << choice;
  return o.str();
}
void ProfileIndex::record(const std::string& k, double v) {
  auto it = d.find(k);
  if (it == d.end() || v < it->second) d[k] = v;
}

static bool better(double v, double best, bool have) { return !have || v < best * (1.0 - TOL); }

struct Node {
  virtual ~Node() {}
  virtual void collect(std::vector<int>& avs) const = 0;
  // exploration protocol (one exploration in flight per node)
  virtual void start(const Config& base, int ctx, ProfileIndex* idx) = 0;
  virtual bool propose(Config& out) = 0;
  virtual void feed(const Metrics& m) = 0;
  virtual void result(Config& into) const = 0;  // writes this subtree's best AVs into `into`
};

struct Leaf : Node {
  int av = 0, n = 1, metric = 0;
  std::string name;
  std::vector<int> n_ctx;
  Config base;
  int ctx = -1, k = 0, nopt = 0, best = 0;
  double bm = 0;
  bool have = false;
  ProfileIndex* idx = nullptr;
  int options(int c) const { return (!n_ctx.empty() && c >= 0) ? n_ctx.at(c) : n; }
  void collect(std::vector<int>& avs) const override { avs.push_back(av); }
  void start(const Config& b, int c, ProfileIndex* ix) override {
    base = b; ctx = c; k = 0; nopt = options(c); have = false; best = 0; idx = ix;
  }
  bool propose(Config& out) override {
    if (k >= nopt) return false;
    out = base;
    out[av] = k;
    return true;
  }
  void feed(const Metrics& m) override {
    const double v = m.at(metric);
    idx->record(ProfileIndex::key(ctx < 0 ? 0 : ctx, name, std::to_string(k), idx->bucket), v);
    if (better(v, bm, have)) { best = k; bm = v; have = true; }
    ++k;
  }
  void result(Config& into) const override { into[av] = best; }
};

struct Exh : Node {
  int metric = 0;
  std::vector<Leaf*> kids;  // owned by `own`
  std::vector<NodeP> own;
  Config base;
  int ctx = -1;
  std::vector<int> combo, nopt, best;
  bool have = false, finished = false;
  double bm = 0;
  ProfileIndex* idx = nullptr;
  void collect(std::vector<int>& avs) const override { for (auto* l : kids) avs.push_back(l->av); }
  void start(const Config& b, int c, ProfileIndex* ix) override {
    base = b; ctx = c; idx = ix; have = false; finished = false;
    nopt.clear();
    for (auto* l : kids) nopt.push_back(l->options(c));
    combo.assign(kids.size(), 0);
    best = combo;
  }
  bool propose(Config& out) override {
    if (finished) return false;
    out = base;
    for (size_t i = 0; i < kids.size(); ++i) out[kids[i]->av] = combo[i];
    return true;
  }
  void feed(const Metrics& m) override {
    const double v = m.at(metric);
    std::string nm, ch;
    for (size_t i = 0; i < kids.size(); ++i) {
      nm += (i ? "+" : "") + kids[i]->name;
      ch += (i ? "," : "") + std::to_string(combo[i]);
    }
    idx->record(ProfileIndex::key(ctx < 0 ? 0 : ctx, nm, ch, idx->bucket), v);
    if (better(v, bm, have)) { best = combo; bm = v; have = true; }
    // advance: last child varies fastest (itertools.product order)
    int i = (int)kids.size() - 1;
    while (i >= 0) {
      if (++combo[i] < nopt[i]) break;
      combo[i] = 0;
      --i;
    }
    if (i < 0) finished = true;
  }
  void result(Config& into) const override {
    for (size_t i = 0; i < kids.size(); ++i) into[kids[i]->av] = best[i];
  }
};

struct Par : Node {
  std::vector<NodeP> kids;
  Config base;
  std::vector<bool> pending;
  std::vector<Config> prop;
  std::vector<std::vector<int>> kid_avs;
  void collect(std::vector<int>& avs) const override { for (auto& k : kids) k->collect(avs); }
  void start(const Config& b, int c, ProfileIndex* ix) override {
    base = b;
    pending.assign(kids.size(), false);
    prop.assign(kids.size(), Config());
    kid_avs.assign(kids.size(), {});
    for (size_t i = 0; i < kids.size(); ++i) {
      kids[i]->collect(kid_avs[i]);
      kids[i]->start(b, c, ix);
      pending[i] = kids[i]->propose(prop[i]);
    }
  }
  bool propose(Config& out) override {
    bool any = false;
    for (bool p : pending) any |= p;
    if (!any) return false;
    out = base;
    for (size_t i = 0; i < kids.size(); ++i) {
      if (pending[i]) {
        for (int a : kid_avs[i]) out[a] = prop[i][a];
      } else {
        kids[i]->result(out);
      }
    }
    return true;
  }
  void feed(const Metrics& m) override {
    for (size_t i = 0; i < kids.size(); ++i) {
      if (!pending[i]) continue;
      kids[i]->feed(m);
      pending[i] = kids[i]->propose(prop[i]);
    }
  }
  void result(Config& into) const override { for (auto& k : kids) k->result(into); }
};

struct Pre : Node {
  std::vector<NodeP> kids;
  Config cur, prop;
  size_t at = 0;
  int ctx = -1;
  ProfileIndex* idx = nullptr;
  bool have_prop = false;
  void collect(std::vector<int>& avs) const override { for (auto& k : kids) k->collect(avs); }
  void advance() {
    while (at < kids.size()) {
      if (kids[at]->propose(prop)) { have_prop = true; return; }
      kids[at]->result(cur);
      ++at;
      if (at < kids.size()) kids[at]->start(cur, ctx, idx);
    }
    have_prop = false;
  }
  void start(const Config& b, int c, ProfileIndex* ix) override {
    cur = b; ctx = c; idx = ix; at = 0;
    if (!kids.empty()) kids[0]->start(cur, ctx, idx);
    advance();
  }
  bool propose(Config& out) override {
    if (!have_prop) return false;
    out = prop;
    return true;
  }
  void feed(const Metrics& m) override {
    kids[at]->feed(m);
    advance();
  }
  void result(Config& into) const override {
    // children < at have their best folded into cur; all children finished when converged
    for (auto& k : kids) k->result(into);
  }
};

struct Fork : Node {
  NodeP ctxleaf_own;
  Leaf* ctxleaf = nullptr;
  NodeP child;
  int metric = 0, reps = 1;
  Config base;
  ProfileIndex* idx = nullptr;
  int cv = 0, phase = 0, rc = 0, rep = 0, best = 0;
  double cur_min = 0, bm = 0;
  bool have = false;
  std::vector<Config> per_ctx;
  void collect(std::vector<int>& avs) const override {
    avs.push_back(ctxleaf->av);
    child->collect(avs);
  }
  void start_ctx() {
    Config b = base;
    b[ctxleaf->av] = cv;
    child->start(b, cv, idx);
  }
  void start(const Config& b, int, ProfileIndex* ix) override {
    base = b; idx = ix; cv = 0; phase = 0; rc = 0; rep = 0; have = false;
    per_ctx.clear();
    start_ctx();
  }
  bool propose(Config& out) override {
    if (phase == 0) {
      while (true) {
        if (child->propose(out)) return true;
        Config r = base;
        child->result(r);
        r[ctxleaf->av] = cv;
        per_ctx.push_back(r);
        if (++cv < ctxleaf->n) { start_ctx(); continue; }
        phase = 1;
        rc = 0; rep = 0;
        break;
      }
    }
    if (phase == 1 && rc < (int)per_ctx.size()) {
      out = per_ctx[rc];
      return true;
    }
    return false;
  }
  void feed(const Metrics& m) override {
    if (phase == 0) { child->feed(m); return; }
    const double v = m.at(metric);
    cur_min = rep == 0 ? v : std::min(cur_min, v);
    if (++rep < reps) return;
    idx->record(ProfileIndex::key(rc, "race", std::to_string(rc), idx->bucket), cur_min);
    if (better(cur_min, bm, have)) { best = rc; bm = cur_min; have = true; }
    rep = 0;
    ++rc;
  }
  void result(Config& into) const override {
    const Config& r = per_ctx.at(best);
    std::vector<int> avs;
    collect(avs);
    for (int a : avs) into[a] = r[a];
  }
};

// ------------------------------------------------------------------------ parser
namespace {
struct Lexer {
  const std::string& s;
  size_t p = 0;
  explicit Lexer(const std::string& str) : s(str) {}
  void ws() { while (p < s.size() && std::isspace((unsigned char)s[p])) ++p; }
  bool peek(char c) { ws(); return p < s.size() && s[p] == c; }
  void expect(char c) {
    ws();
    if (p >= s.size() || s[p] != c) throw std::runtime_error(std::string("tree parse: expected '") + c + "'");
    ++p;
  }
  std::string atom() {
    ws();
    size_t b = p;
    while (p < s.size() && !std::isspace((unsigned char)s[p]) && s[p] != '(' && s[p] != ')') ++p;
    if (b == p) throw std::runtime_error("tree parse: expected atom");
    return s.substr(b, p - b);
  }
};

NodeP parse_node(Lexer& L, Tree& t);

std::unique_ptr<Leaf> parse_leaf_body(Lexer& L, Tree& t) {
  auto l = std::make_unique<Leaf>();
  l->name = L.atom();
  l->n = std::stoi(L.atom());
  if (l->n < 1) throw std::runtime_error("tree parse: leaf needs n >= 1");
  l->metric = t.metric_index(L.atom());
  while (!L.peek(')')) l->n_ctx.push_back(std::stoi(L.atom()));
  l->av = (int)t.avs.size();
  t.avs.push_back(l->name);
  t.av_n.push_back(l->n);
  return l;
}

NodeP parse_node(Lexer& L, Tree& t) {
  L.expect('(');
  const std::string kind = L.atom();
  NodeP out;
  if (kind == "leaf") {
    out = parse_leaf_body(L, t);
  } else if (kind == "exh") {
    auto e = std::make_unique<Exh>();
    e->metric = t.metric_index(L.atom());
    while (!L.peek(')')) {
      L.expect('(');
      if (L.atom() != "leaf") throw std::runtime_error("tree parse: exh children must be leaves");
      auto l = parse_leaf_body(L, t);
      L.expect(')');
      e->kids.push_back(l.get());
      e->own.push_back(std::move(l));
    }
    out = std::move(e);
  } else if (kind == "par" || kind == "pre") {
    std::vector<NodeP> kids;
    while (!L.peek(')')) kids.push_back(parse_node(L, t));
    if (kind == "par") { auto n = std::make_unique<Par>(); n->kids = std::move(kids); out = std::move(n); }
    else { auto n = std::make_unique<Pre>(); n->kids = std::move(kids); out = std::move(n); }
  } else if (kind == "fork") {
    auto f = std::make_unique<Fork>();
    L.expect('(');
    if (L.atom() != "leaf") throw std::runtime_error("tree parse: fork context must be a leaf");
    auto l = parse_leaf_body(L, t);
    L.expect(')');
    f->ctxleaf = l.get();
    f->ctxleaf_own = std::move(l);
    f->metric = t.metric_index(L.atom());
    f->child = parse_node(L, t);
    if (!L.peek(')')) f->reps = std::stoi(L.atom());
    out = std::move(f);
  } else {
    throw std::runtime_error("tree parse: unknown node '" + kind + "'");
  }
  L.expect(')');
  return out;
}
}  // namespace

Tree::Tree() {}
Tree::~Tree() {}
Tree::Tree(Tree&&) noexcept = default;
Tree& Tree::operator=(Tree&&) noexcept = default;

int Tree::av_index(const std::string& n) const {
  for (size_t i = 0; i < avs.size(); ++i) if (avs[i] == n) return (int)i;
  return -1;
}
int Tree::metric_index(const std::string& n) {
  for (size_t i = 0; i < metrics.size(); ++i) if (metrics[i] == n) return (int)i;
  metrics.push_back(n);
  return (int)metrics.size() - 1;
}

Tree parse(const std::string& s) {
  Tree t;
  Lexer L(s);
  t.root = parse_node(L, t);
  L.ws();
  if (L.p != s.size()) throw std::runtime_error("tree parse: trailing input");
  return t;
}

// ------------------------------------------------------------------------ wirer
Wirer::Wirer(Tree* t) : tree_(t) {}
Wirer::~Wirer() {}

void Wirer::start() {
  Config base(tree_->avs.size(), 0);
  tree_->root->start(base, -1, &index_);
  done_ = false;
  trials_ = 0;
  have_prop_ = tree_->root->propose(prop_);
  if (!have_prop_) {
    done_ = true;
    final_ = base;
    tree_->root->result(final_);
  }
}

bool Wirer::propose(Config& out) {
  if (done_ || !have_prop_) return false;
  out = prop_;
  return true;
}

void Wirer::feed(const Metrics& m) {
  if (done_) return;
  ++trials_;
  tree_->root->feed(m);
  have_prop_ = tree_->root->propose(prop_);
  if (!have_prop_) {
    done_ = true;
    final_.assign(tree_->avs.size(), 0);
    tree_->root->result(final_);
  }
}

Config Wirer::final_config() const { return final_; }

}  // namespace tuner
}  // namespace astra
