// L2 tuner: Astra's enumerator output (an update tree of adaptive variables) and the custom wirer
// that explores it online, one configuration per real training step (§4.4-§4.7).
//
//   - AdaptiveVar: a leaf with n options; option 0 is the default (initialize),
//     iterate = next option, get_profile_value = its region metric.
//   - Modes: Par (independent children explored in the same mini-batch),
//     Exh (brute force), Pre (prefix / epoch order), Fork (hierarchical context such as
//     the memory-allocation strategy, explored per context then raced end to end).
//   - ProfileIndex: mangled key "ctx=..|b=..|se=..|node=..|choice=.." → min metric;
//     a changed prefix is a miss.
//   - Tie rule (reading R20): a later option replaces the incumbent only if faster by > 0.5 %.
#pragma once
#include <map>
#include <memory>
#include <string>
#include <vector>

namespace astra {
namespace tuner {

constexpr double TOL = 0.005;

using Config = std::vector<int>;      // one option index per AV (tree order)
using Metrics = std::vector<double>;  // one value per metric (tree order)

struct ProfileIndex {
  std::map<std::string, double> d;
  int bucket = 0;   // key prefix "b=": the input-size bucket this index explores
  static std::string key(int ctx, const std::string& node, const std::string& choice, int bucket = 0, int se = 0);
  void record(const std::string& k, double v);
};

struct Node;
using NodeP = std::unique_ptr<Node>;

struct Tree {
  Tree();
  ~Tree();
  Tree(Tree&&) noexcept;
  Tree& operator=(Tree&&) noexcept;
  NodeP root;
  std::vector<std::string> avs;      // AV names in tree order
  std::vector<int> av_n;             // option counts (context-free)
  std::vector<std::string> metrics;  // metric names in order of first appearance
  int av_index(const std::string& n) const;
  int metric_index(const std::string& n);  // adds if absent
};

// Parse "(par (leaf a 3 m) (exh g (leaf f 3 g) (leaf k 2 g)) (pre ...) (fork (leaf alloc 2 step) step CHILD [reps]))".
Tree parse(const std::string& s);

// The custom wirer: drives exploration of a tree.  Usage:
//   Wirer w(tree); w.start(); while (w.propose(cfg)) { run cfg; w.feed(metrics); } final = w.final_config();
class Wirer {
 public:
  explicit Wirer(Tree* t);
  ~Wirer();
  void start();
  bool propose(Config& out);  // false once converged
  void feed(const Metrics& m);
  Config final_config() const;
  bool converged() const { return done_; }
  int trials() const { return trials_; }
  ProfileIndex& index() { return index_; }

 private:
  Tree* tree_;
  ProfileIndex index_;
  bool done_ = false;
  bool have_prop_ = false;
  Config prop_;
  int trials_ = 0;
  Config final_;
};

}  // namespace tuner
}  // namespace astra
