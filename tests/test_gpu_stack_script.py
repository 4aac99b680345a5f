"""SURVEY §4 T3 on the device: the paper's worked examples of the two-level stack (Fig 2) and of
the two steals (Fig 3), replayed on the walker kernel's OWN stack code (dfs_debug_stack_script:
the push / pop / flush / refill / Alg 3 / Alg 4 lambdas the traversal uses), with the values
printed in the paper (tests/golden/*.json, cited per case).

Conventions: the kernel's head/tail are monotone 16-bit counters (slot = counter mod H); the
paper's pointers are those counters mod hot_size.  hot_size = 4 with capacity 3 is the kernel's
ring_cap = 3 (full <=> 3 entries, batch = (cap + 1) / 2 = 2).  Vertex ids a, b, c = 10, 11, 12.
"""
import json
import os

import numpy as np
import pytest

import graphgen

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_ppopp_niul0c26_b200 import Graph, Options

GOLD = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")
A, B, C = 10, 11, 12
END, SET, RING, COLD, PUSH, POP, FLUSH, REFILL, STEAL_INTRA, STEAL_INTER, DUMP, READ_RING, READ_COLD = range(13)


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


@pytest.fixture(scope="module")
def G():
    g = graphgen.grid(64, 64)
    with Graph(g.row_ptr, g.col_idx) as h:
        yield h


@pytest.mark.parametrize("lanes", [16, 8, 4, 2])
def test_fig2_two_level_stack_on_kernel_code(G, lanes):
    d = _gold("fig2_two_level_stack.json")
    hs = d["hot_size"]
    o = Options(ring_cap=hs - 1)
    cases = {c["op"]: c for c in d["cases"]}
    # (c) push <a|i> at head 0 (tail 2): counters tail = 2, head = 4 (= 0 mod 4)
    c = cases["push"]
    out = G.stack_script(lanes, [(SET, 0, 4, c["before"]["tail"], 0, 0), (PUSH, 0, A, 7), (DUMP, 0),
                                 (READ_RING, 0, 4)], options=o)
    head, tail = out[0], out[1]
    assert (head % hs, tail % hs) == (c["after"]["head"], c["after"]["tail"]), c["cite"]
    assert (4 % hs) == c["slot"] and tuple(out[4:6]) == (A, 7)
    # (d) pop at head 0 (tail 1): counters tail = 1, head = 4; the entry at counter 3 comes back
    c = cases["pop"]
    out = G.stack_script(lanes, [(SET, 0, 4, c["before"]["tail"], 0, 0), (RING, 0, 3, A, -1), (POP, 0), (DUMP, 0)],
                         options=o)
    assert tuple(out[0:2]) == (A, -1)
    assert (out[2] % hs, out[3] % hs) == (c["after"]["head"], c["after"]["tail"]), c["cite"]
    assert 3 % hs == c["slot"]
    # (e) flush when full: head 1, tail 2 (3 entries = capacity): counters tail = 2, head = 5
    c = cases["flush"]
    b = c["before"]
    out = G.stack_script(lanes, [(SET, 0, 5, b["tail"], b["top"], b["bottom"]), (RING, 0, 2, A, 1), (RING, 0, 3, B, 2),
                                 (RING, 0, 4, C, 3), (FLUSH, 0, 2, 0), (DUMP, 0), (READ_COLD, 0, 2), (READ_COLD, 0, 3)],
                         options=o)
    hd, tl, top, bot = out[0:4]
    a = c["after"]
    assert (hd % hs, tl % hs, top, bot) == (a["head"], a["tail"], a["top"], a["bottom"]), c["cite"]
    assert [2 % hs, 3 % hs] == c["moved_from_slots"] and [2, 3] == c["moved_to_positions"]
    assert tuple(out[4:8]) == (A, 1, B, 2)                  # oldest entries, in order
    # (f) refill when empty: head = tail = 1, ColdSeg [1, 5): positions 3, 4 come back at slots 1, 2
    c = cases["refill"]
    b = c["before"]
    out = G.stack_script(lanes, [(SET, 0, b["head"], b["tail"], b["top"], b["bottom"]), (COLD, 0, 3, A, 1),
                                 (COLD, 0, 4, B, 2), (REFILL, 0), (DUMP, 0), (READ_RING, 0, 1), (READ_RING, 0, 2)],
                         options=o)
    assert out[0] == 2                                      # batch = 2 entries moved
    a = c["after"]
    assert (out[1] % hs, out[2] % hs, out[3], out[4]) == (a["head"], a["tail"], a["top"], a["bottom"]), c["cite"]
    assert c["moved_to_slots"] == [1, 2] and c["moved_from_positions"] == [3, 4]
    assert tuple(out[5:9]) == (A, 1, B, 2)


@pytest.mark.parametrize("lanes", [8, 4, 2])              # >= 3 walkers per warp
def test_fig3a_intra_block_steal_on_kernel_code(G, lanes):
    d = _gold("fig3_steals.json")["intra"]
    e = d["expect"]
    o = Options(hot_cutoff=d["hot_cutoff"], steal_half=False)
    w = d["warps"]
    winner, loser = d["thieves"]
    out = G.stack_script(lanes, [
        (SET, 0, w["0"]["head"], w["0"]["tail"], 0, 0), (RING, 0, 0, A, 1), (RING, 0, 1, B, 2),
        (SET, 1, w["1"]["head"], w["1"]["tail"], 0, 0), (SET, 2, w["2"]["head"], w["2"]["tail"], 0, 0),
        (STEAL_INTRA, 1 << winner), (DUMP, 0), (DUMP, winner), (READ_RING, winner, 0),
        (STEAL_INTRA, 1 << loser), (DUMP, loser)], options=o)
    assert out[0] == 1 << winner                            # Warp1 (walker 1) received the entry
    v_head, v_tail = out[1], out[2]
    assert v_tail == e["victim_tail_after"] and v_head - v_tail == e["loser_sees_rest"], d["cite"]
    assert out[5] == e["winner_head_after"]
    assert tuple(out[9:11]) == (A, 1)                       # copies <a|1>
    assert out[11] == 0                                     # Warp2: rest 1 < hot_cutoff 2, no steal
    assert out[12] == 0 and out[13] == 0                    # its ring stays empty
    assert e["mask_before"] == "100" and e["mask_after"] == "110"   # (walker 1 became active)


@pytest.mark.parametrize("lanes", [8, 4, 2])
def test_fig3b_inter_block_steal_on_kernel_code(G, lanes):
    d = _gold("fig3_steals.json")["inter"]
    e = d["expect"]
    o = Options(cold_cutoff=d["cold_cutoff"], steal_half=False)
    vw = d["victim_block_warps"]
    thief = 3
    out = G.stack_script(lanes, [
        (SET, 0, 0, 0, vw["0"]["top"], vw["0"]["bottom"]), (SET, 1, 0, 0, vw["1"]["top"], vw["1"]["bottom"]),
        (COLD, 1, 0, A, 2), (COLD, 1, 1, C, 1), (COLD, 1, 2, B, 3), (COLD, 1, 3, B, 4),
        (SET, 2, 0, 0, vw["2"]["top"], vw["2"]["bottom"]), (SET, thief, 0, 0, 0, 0),
        (STEAL_INTER, 1 << thief), (DUMP, e["victim_warp"]), (DUMP, thief), (READ_RING, thief, 0),
        (READ_RING, thief, 1)], options=o)
    assert out[0] == 1 << thief, d["cite"]
    top, bot = out[3], out[4]
    assert bot == e["bottom_after"] and top - bot == e["victim_rest_after"]
    assert out[5] == e["thief_head_after"] and out[5] - out[6] == e["stolen"]
    assert tuple(out[9:13]) == (A, 2, C, 1)                 # copies <a|2>, <c|1> from the bottom
