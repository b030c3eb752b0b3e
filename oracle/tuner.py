"""Plain model of Astra's online exploration (custom wirer) on an injected cost table.

TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Follows PAPER.md §4.4.2-§4.7 step by step:
* adaptive variables with initialize / iterate / get_profile_value: `Leaf`;
  option 0 is the default ("initialize: Reset to default choice");
* the update tree with modes Parallel / Exhaustive / Prefix: `Par`, `Exh`, `Pre`;
* parallel exploration: independent children iterate in the same mini-batch; trials =
  max over children (worked example 5 groups × (3 fusion × 2 kernels) → 6 trials
  instead of (3·2)^5 = 7776);
* hierarchical exploration: a top-level fork over a context variable (memory allocation
  strategy); the subtree is explored per context with keys prefixed by the context, then
  the best configuration of every context is raced end to end: `Fork`;
* prefix exploration: child k explored with children < k frozen at their best, later ones
  at default; cost additive: `Pre`;
* equivalence exploration: m equivalent kernels on 2 streams → only the split count
  matters, k ∈ {1..⌊m/2⌋} ("2^10 → 5"): `equivalence_options`;
* profile index keyed by mangled keys; a changed prefix is a miss: `ProfileIndex`.

Readings: R19 one measurement per configuration on the fake clock (the live
tuner takes the minimum over k interleaved reps); R20 ties: a later option replaces the
incumbent only if it is faster by more than `TOL` (relative), so the lower enumeration index
wins within 0.5%; R22 equivalence counts unordered non-empty 2-stream splits.
Each trial is one real training mini-batch (work-conserving, P:9).
"""
from __future__ import annotations

import itertools
import math

TOL = 0.005


class Leaf:
    """An adaptive variable with `n` options (or a per-context count `n_ctx[c]`)."""

    def __init__(self, name, n, metric, n_ctx=None):
        self.name, self.n, self.metric, self.n_ctx = name, n, metric, n_ctx

    def avs(self):
        return [self.name]

    def options(self, ctx):
        if self.n_ctx is not None and ctx is not None:
            return self.n_ctx[ctx]
        return self.n


class Exh:
    """Exhaustive (brute-force) product over leaf children; metric = the node metric."""

    def __init__(self, metric, *children):
        self.metric, self.children = metric, list(children)

    def avs(self):
        return [a for c in self.children for a in c.avs()]


class Par:
    def __init__(self, *children):
        self.children = list(children)

    def avs(self):
        return [a for c in self.children for a in c.avs()]


class Pre:
    def __init__(self, *children):
        self.children = list(children)

    def avs(self):
        return [a for c in self.children for a in c.avs()]


class Fork:
    """Hierarchical fork over context variable `ctx` (a Leaf); final race on `metric`."""

    def __init__(self, ctx, child, metric, reps=1):
        self.ctx, self.child, self.metric, self.reps = ctx, child, metric, reps

    def avs(self):
        return [self.ctx.name] + self.child.avs()


def equivalence_options(m, streams=2):
    """Unordered non-empty splits of m equivalent kernels over 2 streams: k ∈ {1..⌊m/2⌋}."""
    assert streams == 2
    return list(range(1, m // 2 + 1))


class ProfileIndex:
    """Mangled key → minimum metric seen."""

    def __init__(self):
        self.d = {}

    @staticmethod
    def key(ctx, node, choice, bucket=0, se=0):
        return f"ctx={ctx}|b={bucket}|se={se}|node={node}|choice={choice}"

    def record(self, k, v):
        self.d[k] = min(v, self.d.get(k, math.inf))

    def __contains__(self, k):
        return k in self.d


def _better(v, best):
    return best is None or v < best * (1.0 - TOL)


def _explore(node, base, ctx, index):
    """Generator: yields full configs (dicts), receives metric dicts, returns best sub-assignment."""
    if isinstance(node, Leaf):
        best, bm = None, None
        for o in range(node.options(ctx)):
            cfg = dict(base)
            cfg[node.name] = o
            m = yield cfg
            v = m[node.metric]
            index.record(ProfileIndex.key(ctx, node.name, o), v)
            if _better(v, bm):
                best, bm = o, v
        return {node.name: best}
    if isinstance(node, Exh):
        ranges = [range(c.options(ctx)) for c in node.children]
        best, bm = None, None
        for combo in itertools.product(*ranges):           # first child varies slowest
            cfg = dict(base)
            for c, o in zip(node.children, combo):
                cfg[c.name] = o
            m = yield cfg
            v = m[node.metric]
            index.record(ProfileIndex.key(ctx, "+".join(c.name for c in node.children),
                                          ",".join(map(str, combo))), v)
            if _better(v, bm):
                best, bm = combo, v
        return {c.name: o for c, o in zip(node.children, best)}
    if isinstance(node, Par):
        gens = [_explore(c, base, ctx, index) for c in node.children]
        held = [None] * len(gens)        # best sub-assignment once a child is done
        pending = [None] * len(gens)     # the config a live child wants to try
        for k, g in enumerate(gens):
            try:
                pending[k] = next(g)
            except StopIteration as e:
                held[k] = e.value
        while any(p is not None for p in pending):
            cfg = dict(base)
            for k, c in enumerate(node.children):
                src = pending[k] if pending[k] is not None else held[k]
                for a in c.avs():
                    cfg[a] = src[a]
            m = yield cfg
            for k, g in enumerate(gens):
                if pending[k] is None:
                    continue
                try:
                    pending[k] = g.send(m)
                except StopIteration as e:
                    pending[k], held[k] = None, e.value
        out = {}
        for h in held:
            out.update(h)
        return out
    if isinstance(node, Pre):
        cur = dict(base)
        out = {}
        for c in node.children:
            best = yield from _explore(c, cur, ctx, index)
            cur.update(best)
            out.update(best)
        return out
    if isinstance(node, Fork):
        per_ctx = []
        for cv in range(node.ctx.n):
            b = dict(base)
            b[node.ctx.name] = cv
            best = yield from _explore(node.child, b, cv, index)
            per_ctx.append(dict(best, **{node.ctx.name: cv}))
        best, bm = None, None
        for cv, cfg_best in enumerate(per_ctx):
            cfg = dict(base)
            cfg.update(cfg_best)
            v = math.inf
            for _ in range(node.reps):
                m = yield cfg
                v = min(v, m[node.metric])
            index.record(ProfileIndex.key(cv, "race", cv), v)
            if _better(v, bm):
                best, bm = cv, v
        return per_ctx[best]
    raise TypeError(node)


def defaults(tree):
    return {a: 0 for a in tree.avs()}


def run(tree, cost):
    """Drive exploration to convergence.  cost(config) -> {metric: value}.

    Returns (trials, final_config, index): `trials` is the list of configs run, one per
    mini-batch; `final_config` the converged configuration.
    """
    index = ProfileIndex()
    gen = _explore(tree, defaults(tree), None, index)
    trials = []
    try:
        cfg = next(gen)
        while True:
            trials.append(cfg)
            cfg = gen.send(cost(cfg))
    except StopIteration as e:
        final = defaults(tree)
        final.update(e.value)
        return trials, final, index


def brute_force(tree, cost, metric):
    """Argmin of `metric` over the full product space (for separable toy spaces)."""
    avs = tree.avs()
    leaves = {}

    def collect(n):
        if isinstance(n, Leaf):
            leaves[n.name] = n
        elif isinstance(n, Fork):
            leaves[n.ctx.name] = n.ctx
            collect(n.child)
        else:
            for c in n.children:
                collect(c)
    collect(tree)
    best, bm = None, None
    for combo in itertools.product(*[range(leaves[a].n) for a in avs]):
        cfg = dict(zip(avs, combo))
        v = cost(cfg)[metric]
        if bm is None or v < bm:
            best, bm = cfg, v
    return best, bm
