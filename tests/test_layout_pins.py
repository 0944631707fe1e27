"""Pins of the layout-side oracle helpers (oracle/layout_oracle.py) against the paper's worked
examples: Fig. 1 reorg order and the Tree #2 swap, Fig. 3 SimHash / LSH
(P:648-769), and the probability identities of P:399-406."""
import hashlib
import json
import os

import numpy as np

import gen
import oracle
from oracle import layout_oracle as lo
from tlib import GOLDEN


def test_fig1_reorg_order():
    g = json.load(open(os.path.join(GOLDEN, "fig1_reorg.json")))
    levels = lo.reorg_order(g["trees"])
    assert levels[0] == g["level1"]
    assert levels[1] == g["level2"]
    assert levels[2] == g["level3"]


def _fig1_forest():
    """Fig. 1 trees as node arrays; names -> ids; features F1..F7 -> 0..6 (tree #1 tests F1..F7
    per SURVEY W2'); thresholds 0.5."""
    g = json.load(open(os.path.join(GOLDEN, "fig1_reorg.json")))
    names, feature, left, right = [], [], [], []
    roots = []
    for t in g["trees"]:
        order = [t["_root"]]
        i = 0
        while i < len(order):
            if order[i] in t:
                order += t[order[i]]
            i += 1
        roots.append(len(names))
        names += order
    idx = {n: i for i, n in enumerate(names)}
    adj = {}
    for t in g["trees"]:
        adj.update({k: v for k, v in t.items() if k != "_root"})
    for i, n in enumerate(names):
        if n in adj:
            feature.append(int(n[2]) - 1 if n[1] == "1" else i % 7)
            left.append(idx[adj[n][0]])
            right.append(idx[adj[n][1]])
        else:
            feature.append(-1); left.append(-1); right.append(-1)
    forest = dict(root=np.array(roots, np.int32), feature=np.array(feature, np.int32),
                  threshold=np.full(len(names), 0.5, np.float32), left=np.array(left, np.int32),
                  right=np.array(right, np.int32), leaf_value=np.zeros(len(names), np.float32),
                  default_left=None, tree_class=None)
    return g, names, idx, forest


def test_fig1_swap_rule_and_reorg_after_swap():
    g, names, idx, forest = _fig1_forest()
    counts = np.zeros(len(names), np.uint64)
    for r in forest["root"]:
        counts[r] = 100
    for e, c in g["edge_counts_after_training"].items():
        counts[idx[e.split("->")[1]]] = c
    # unreached subtrees of tree 3 keep zero counts => no swap there (reading Z5)
    hl = lo.hot_is_left(forest, counts)
    assert hl[idx["V21"]] == 0          # 0.3 vs 0.7 => swapped
    assert hl[idx["V11"]] == 1 and hl[idx["V12"]] == 1
    assert hl[idx["V13"]] == 0          # 0.3 vs 0.7 (Fig. 1 labels; Fig. 3 token order 3-7, 3-6)
    # reorg order after applying the swaps: children listed hot first
    trees = []
    for t in g["trees"]:
        tt = {"_root": t["_root"]}
        for k, v in t.items():
            if k == "_root":
                continue
            tt[k] = v if hl[idx[k]] else v[::-1]
        trees.append(tt)
    lv = lo.reorg_order(trees)
    assert lv[1][1] == "V23"            # V23 moved to the first (hot) slot of tree #2
    assert lv[2][0:3] == g["after_swap_level3_pos4"]   # "V25 ... and V14 ... contiguous"


def test_fig3_simhash_checksum_and_normalisation():
    g = json.load(open(os.path.join(GOLDEN, "fig3_simhash.json")))
    cs, bits = lo.simhash(np.array(g["strings"]), np.array(g["weights"]))
    assert np.allclose(cs, g["checksum"], atol=1e-12)
    assert bits.tolist() == g["normalized"]
    assert bits.tolist() == g["reps"]["T1"]


def test_fig3_lsh_collisions_groups_and_order():
    g = json.load(open(os.path.join(GOLDEN, "fig3_simhash.json")))
    names = ["T1", "T2", "T3"]
    bits = np.array([g["reps"][n] for n in names], np.uint8)
    col = lo.lsh_collisions(bits, g["m_chunks"])
    assert col[0, 1] == g["collisions"]["T1&T2"]
    assert col[1, 2] == g["collisions"]["T2&T3"]
    assert col[0, 2] == g["collisions"]["T1&T3"]
    w = bits.shape[1] // g["m_chunks"]
    for c, groups in enumerate(g["chunk_groups"]):
        keys = [lo.rabin_karp(bits[t, c * w:(c + 1) * w]) for t in range(3)]
        got = {frozenset(names[t] for t in range(3) if keys[t] == keys[s]) for s in range(3)}
        assert got == {frozenset(x) for x in groups}
    assert [names[t] for t in lo.lsh_order(col)] == g["order"]


def test_fig3_tokens_and_weights_from_fig1_probabilities():
    g3 = json.load(open(os.path.join(GOLDEN, "fig3_simhash.json")))
    g, names, idx, forest = _fig1_forest()
    counts = np.zeros(len(names), np.uint64)
    for r in forest["root"]:
        counts[r] = 100
    for e, c in g["edge_counts_after_training"].items():
        counts[idx[e.split("->")[1]]] = c
    hl = lo.hot_is_left(forest, counts)
    toks = lo.tokens(forest, 0, 2, hl)
    assert [[names[k] for k in t] for t in toks] == g3["tree1_tokens_tnodes2"]
    ep = lo.edge_probabilities(forest, counts)
    npb = lo.node_probabilities(forest, ep)
    w = [round(npb[t[-1]], 12) for t in toks]
    assert w == g3["weights"]


def test_node_probability_is_product_of_edge_probabilities():
    f = gen.make_forest(2, n_trees=25)
    Xc = gen.make_calibration(2, 4000)
    cnt = oracle.node_counts(f, Xc)
    ep = lo.edge_probabilities(f, cnt)
    npb = lo.node_probabilities(f, ep)
    assert np.allclose(npb, cnt / len(Xc), rtol=1e-12, atol=1e-15)
    # leaf probabilities of each tree sum to 1 (one path per sample)
    leaves = f["feature"] < 0
    bounds = np.append(f["root"], len(f["feature"]))
    for t in range(25):
        s = npb[bounds[t]:bounds[t + 1]][leaves[bounds[t]:bounds[t + 1]]].sum()
        assert abs(s - 1.0) < 1e-12
    hl = lo.hot_is_left(f, cnt)
    internal = np.nonzero(f["feature"] >= 0)[0]
    hot = np.where(hl[internal] == 1, f["left"][internal], f["right"][internal])
    cold = np.where(hl[internal] == 1, f["right"][internal], f["left"][internal])
    assert (cnt[hot] >= cnt[cold]).all()


def test_token_bits_follow_sha1_msb_first():
    data = b"\x01\x00\x00\x05\x00\xff"
    bits = lo.token_bits(data, 128)
    ref = np.unpackbits(np.frombuffer(hashlib.sha1(data).digest(), np.uint8))[:128]
    assert np.array_equal(bits, ref)
    long = lo.token_bits(data, 256)
    ref2 = np.unpackbits(np.frombuffer(hashlib.sha1(data + b"\x00").digest()
                                       + hashlib.sha1(data + b"\x01").digest(), np.uint8))[:256]
    assert np.array_equal(long, ref2)
