"""Pins for the oracle tuner model against the paper's worked counts and brute force."""
import itertools

import pytest

from oracle import tuner as TU
from helpers import golden

PAPER = golden("paper_worked_examples.json")


def _additive_cost(tables):
    """cost(cfg) -> metrics; each metric is a sum of per-AV table entries (separable)."""
    def cost(cfg):
        out = {}
        for metric, parts in tables.items():
            out[metric] = sum(tab[cfg[av]] for av, tab in parts)
        out["step"] = sum(out[m] for m in tables)
        return out
    return cost


def test_parallel_exploration_worked_example_p220():
    """5 fusion groups × (3 fusion chunkings × 2 kernels): parallel exploration needs 3·2 = 6
    trials; an end-to-end one-at-a-time search over the same space needs (3·2)^5 = 7776."""
    P = PAPER["parallel_exploration"]
    G, NF, NK = P["groups"], P["fusion_choices"], P["kernel_choices"]
    groups = []
    tables = {}
    for gi in range(G):
        fus, ker = TU.Leaf(f"fuse{gi}", NF, f"g{gi}"), TU.Leaf(f"kern{gi}", NK, f"g{gi}")
        groups.append(TU.Exh(f"g{gi}", fus, ker))
        tables[f"g{gi}"] = [(f"fuse{gi}", [5.0 + gi, 3.0, 4.0 - 0.1 * gi]), (f"kern{gi}", [1.0, 0.5 + 0.3 * (gi % 2)])]
    tree = TU.Par(*groups)
    cost = _additive_cost(tables)
    trials, final, _ = TU.run(tree, cost)
    assert len(trials) == P["parallel_trials"]
    # the one-at-a-time search space, counted by enumerating every joint configuration
    full = sum(1 for _ in itertools.product(*[range(NF * NK)] * G))
    assert full == P["mutation_trials"]
    best, _ = TU.brute_force(tree, cost, "step")
    assert final == best


def test_equivalence_exploration_p247():
    """10 equivalent kernels on 2 streams: only the split count matters → 5 choices, not 2^10."""
    P = PAPER["equivalence_exploration"]
    n = P["kernels"]
    assert len(TU.equivalence_options(n)) == P["choices"]
    assert TU.equivalence_options(n) == [1, 2, 3, 4, 5]
    # brute force: distinct unordered non-empty 2-stream splits of n identical kernels, against the
    # 2^n assignments of distinguishable kernels to the streams
    assign = list(itertools.product(range(P["streams"]), repeat=n))
    splits = {tuple(sorted((a.count(0), a.count(1)))) for a in assign if 0 < a.count(0) < n}
    assert len(splits) == P["choices"] and len(assign) == P["naive_space"]


def test_prefix_exploration_is_additive_p243():
    """Prefix over epochs: trials = Σ n_i (not Π n_i); child k sees children < k at their best."""
    ns = [3, 4, 2, 5]
    leaves = [TU.Leaf(f"e{k}", n, f"epoch{k}") for k, n in enumerate(ns)]
    tree = TU.Pre(*leaves)
    # history-sensitive cost: epoch k's metric depends on the choices of epochs ≤ k
    def cost(cfg):
        out, acc = {}, 0.0
        for k, n in enumerate(ns):
            acc += 1.0 + ((cfg[f"e{k}"] * 7 + 3 * k + (cfg[f"e{k-1}"] if k else 0)) % n) * 0.25
            out[f"epoch{k}"] = acc
        out["step"] = acc
        return out
    trials, final, _ = TU.run(tree, cost)
    assert len(trials) == sum(ns)
    prod = 1
    for n in ns:
        prod *= n
    assert prod == 120
    # each epoch's choice is the argmin given the frozen prefix
    frozen = {f"e{k}": 0 for k in range(len(ns))}
    for k in range(len(ns)):
        vals = []
        for o in range(ns[k]):
            c = dict(frozen)
            c[f"e{k}"] = o
            vals.append(cost(c)[f"epoch{k}"])
        frozen[f"e{k}"] = min(range(ns[k]), key=lambda o: (vals[o], o))
    assert final == frozen


def test_hierarchical_fork_restricts_and_races_p226():
    """Fork over an allocation strategy: per-context restricted exploration, then a race of the
    per-context bests end to end; result equals brute force over the valid combinations."""
    alloc = TU.Leaf("alloc", 2, "step")
    fuse = TU.Leaf("fuse", 3, "gemm", n_ctx=[1, 3])        # ctx 0 cannot fuse (non-contiguous)
    kern = TU.Leaf("kern", 2, "kern")
    tree = TU.Fork(alloc, TU.Par(fuse, kern), "step")
    def cost(cfg):
        g = [10.0, 6.0, 7.0][cfg["fuse"]] + (2.0 if cfg["alloc"] == 1 else 0.0)
        k = [3.0, 2.0][cfg["kern"]]
        return {"gemm": g, "kern": k, "step": g + k + (1.0 if cfg["alloc"] == 0 else 0.0)}
    trials, final, idx = TU.run(tree, cost)
    # ctx0: max(1, 2) = 2 trials; ctx1: max(3, 2) = 3 trials; race: 2 trials
    assert len(trials) == 2 + 3 + 2
    assert final == {"alloc": 1, "fuse": 1, "kern": 1}
    # keys of different contexts never alias (a changed prefix is a miss)
    assert TU.ProfileIndex.key(0, "fuse", 0) != TU.ProfileIndex.key(1, "fuse", 0)
    assert TU.ProfileIndex.key(1, "fuse", 1) in idx


def test_tie_rule_prefers_lower_index():
    leaf = TU.Leaf("a", 3, "m")
    trials, final, _ = TU.run(leaf, lambda c: {"m": [1.0, 0.999, 0.5][c["a"]]})
    assert final == {"a": 2}
    trials, final, _ = TU.run(leaf, lambda c: {"m": [1.0, 0.999, 0.998][c["a"]]})
    assert final == {"a": 0}


@pytest.mark.parametrize("seed", range(5))
def test_parallel_matches_brute_force_on_separable_spaces(seed):
    import random
    r = random.Random(seed)
    leaves, tables = [], {}
    for k in range(4):
        n = r.randint(1, 4)
        leaves.append(TU.Leaf(f"v{k}", n, f"m{k}"))
        tables[f"m{k}"] = [(f"v{k}", [r.uniform(1, 2) for _ in range(n)])]
    tree = TU.Par(*leaves)
    cost = _additive_cost(tables)
    trials, final, _ = TU.run(tree, cost)
    best, _ = TU.brute_force(tree, cost, "step")
    assert final == best
    assert len(trials) == max(l.n for l in leaves)
