"""The native (C++) custom wirer against the oracle tuner model on identical update trees and
identical fake-clock cost tables: same trial sequence, same final configuration (bit-exact host
logic).  Also re-checks the paper's worked counts through the native code."""
import random

import pytest

import paper_conf_asplos_sivathanucsz19_b200 as A
from oracle import tuner as TU
from helpers import golden


def _to_sexpr(node):
    if isinstance(node, TU.Leaf):
        extra = (" " + " ".join(map(str, node.n_ctx))) if node.n_ctx else ""
        return f"(leaf {node.name} {node.n} {node.metric}{extra})"
    if isinstance(node, TU.Exh):
        return f"(exh {node.metric} " + " ".join(_to_sexpr(c) for c in node.children) + ")"
    if isinstance(node, TU.Par):
        return "(par " + " ".join(_to_sexpr(c) for c in node.children) + ")"
    if isinstance(node, TU.Pre):
        return "(pre " + " ".join(_to_sexpr(c) for c in node.children) + ")"
    if isinstance(node, TU.Fork):
        return f"(fork {_to_sexpr(node.ctx)} {node.metric} {_to_sexpr(node.child)} {node.reps})"
    raise TypeError(node)


def _metrics_order(node, acc):
    if isinstance(node, TU.Leaf):
        if node.metric not in acc:
            acc.append(node.metric)
    elif isinstance(node, TU.Exh):
        if node.metric not in acc:
            acc.append(node.metric)
        for c in node.children:
            _metrics_order(c, acc)
    elif isinstance(node, TU.Fork):
        _metrics_order(node.ctx, acc)
        if node.metric not in acc:
            acc.append(node.metric)
        _metrics_order(node.child, acc)
    else:
        for c in node.children:
            _metrics_order(c, acc)
    return acc


def _compare(tree, cost):
    trials_py, final_py, _ = TU.run(tree, cost)
    avs = tree.avs()
    metrics = _metrics_order(tree, [])

    def native_cost(cfg_list):
        m = cost(dict(zip(avs, cfg_list)))
        return [m[k] for k in metrics]
    res = A.tuner_selftest(_to_sexpr(tree), native_cost)
    assert res["n_trials"] == len(trials_py)
    assert res["trials"] == [[t[a] for a in avs] for t in trials_py]
    assert res["final"] == [final_py[a] for a in avs]
    return res


def _random_tree(r, depth=0, counter=[0], allow_fork=True):
    kind = r.choice(["leaf", "leaf", "par", "pre", "exh"] + (["fork"] if allow_fork and depth == 0 else []))
    if depth >= 2:
        kind = "leaf"

    def leaf(metric=None):
        counter[0] += 1
        return TU.Leaf(f"v{counter[0]}", r.randint(1, 4), metric or f"m{r.randint(0, 5)}")
    if kind == "leaf":
        return leaf()
    if kind == "exh":
        m = f"m{r.randint(0, 5)}"
        return TU.Exh(m, *[leaf(m) for _ in range(r.randint(1, 3))])
    if kind == "fork":
        counter[0] += 1
        return TU.Fork(TU.Leaf(f"ctx{counter[0]}", r.randint(1, 3), "step"), _random_tree(r, depth + 1, counter, False),
                       "step", r.randint(1, 2))
    kids = [_random_tree(r, depth + 1, counter, False) for _ in range(r.randint(1, 3))]
    return TU.Par(*kids) if kind == "par" else TU.Pre(*kids)


def _random_cost(r, tree):
    avs = tree.avs()
    tables = {(a, o, m): r.uniform(1.0, 2.0) for a in avs for o in range(8) for m in range(6)}
    noise = r.uniform(0, 0.01)

    def cost(cfg):
        out = {}
        for m in range(6):
            out[f"m{m}"] = sum(tables[(a, cfg[a], m)] for a in avs) + noise * m
        out["step"] = sum(out[f"m{m}"] for m in range(6))
        return out
    return cost


@pytest.mark.parametrize("seed", range(40))
def test_native_wirer_equals_oracle_random_trees(seed):
    r = random.Random(seed)
    tree = _random_tree(r, counter=[0])
    _compare(tree, _random_cost(r, tree))


def test_native_parallel_worked_example_p220():
    P = golden("paper_worked_examples.json")["parallel_exploration"]
    groups, tables = [], {}
    for gi in range(P["groups"]):
        groups.append(TU.Exh(f"g{gi}", TU.Leaf(f"fuse{gi}", P["fusion_choices"], f"g{gi}"),
                             TU.Leaf(f"kern{gi}", P["kernel_choices"], f"g{gi}")))
        tables[gi] = ([5.0 + gi, 3.0, 4.0 - 0.1 * gi], [1.0, 0.5 + 0.3 * (gi % 2)])

    def cost(cfg):
        out = {f"g{gi}": tables[gi][0][cfg[f"fuse{gi}"]] + tables[gi][1][cfg[f"kern{gi}"]] for gi in range(P["groups"])}
        return out
    res = _compare(TU.Par(*groups), cost)
    assert res["n_trials"] == P["parallel_trials"]


def test_native_prefix_additive_p243():
    ns = [3, 4, 2, 5]
    tree = TU.Pre(*[TU.Leaf(f"e{k}", n, f"ep{k}") for k, n in enumerate(ns)])

    def cost(cfg):
        acc, out = 0.0, {}
        for k, n in enumerate(ns):
            acc += 1.0 + ((cfg[f"e{k}"] * 7 + 3 * k) % n) * 0.25
            out[f"ep{k}"] = acc
        return out
    res = _compare(tree, cost)
    assert res["n_trials"] == sum(ns)


def test_native_rejects_bad_tree():
    with pytest.raises(A.AstraError):
        A.tuner_selftest("(par (leaf a 0 m))", lambda c: [0.0])
    with pytest.raises(A.AstraError):
        A.tuner_selftest("(bogus)", lambda c: [0.0])
