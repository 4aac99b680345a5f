"""Replay the paper's worked examples (Figs 2 and 3, tests/golden/*.json, cited per case) against
the test-side stack model (tests/stack_model.py) that mirrors the kernel's conventions."""
import json
import os

from tests import stack_model as sm

G = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load(name):
    with open(os.path.join(G, name)) as f:
        return json.load(f)


def test_fig2_two_level_stack_values():
    d = load("fig2_two_level_stack.json")
    hs, batch = d["hot_size"], d["batch_size"]
    for c in d["cases"]:
        b, a = c["before"], c["after"]
        ring = sm.HotRing(hs, b["head"], b["tail"])
        cold = sm.ColdSeg(b.get("top", 0), b.get("bottom", 0))
        if c["op"] == "push":
            slot = ring.push(tuple(c["entry"]))
            assert slot == c["slot"]
        elif c["op"] == "pop":
            assert ring.pop() == c["slot"]
        elif c["op"] == "flush":
            ring.slots[2], ring.slots[3] = ("a", "i"), ("b", "j")
            ring.head = b["head"]
            assert ring.full(), c["cite"]
            moved = ring.flush(cold, batch)
            assert [m[0] for m in moved] == c["moved_from_slots"]
            assert [m[1] for m in moved] == c["moved_to_positions"]
        elif c["op"] == "refill":
            assert ring.head == ring.tail                    # empty
            cold.data = {3: ("a", "i"), 4: ("b", "j")}
            moved = ring.refill(cold, batch)
            assert [m[0] for m in moved] == c["moved_from_positions"]
            assert [m[1] for m in moved] == c["moved_to_slots"]
        got = {"head": ring.head, "tail": ring.tail}
        if "top" in a:
            got.update(top=cold.top, bottom=cold.bottom)
        assert got == a, (c["op"], c["cite"], got)


def test_fig3_intra_block_steal():
    d = load("fig3_steals.json")["intra"]
    rings = {int(k): sm.HotRing(d["hot_size"], v["head"], v["tail"]) for k, v in d["warps"].items()}
    rings[0].slots[0], rings[0].slots[1] = ("a", 1), ("b", 2)
    mask = {0: 1, 1: 0, 2: 0}
    before = "".join(str(mask[i]) for i in range(3))
    winner, loser = d["thieves"]
    victim = sm.intra_steal(rings, mask, winner, d["hot_cutoff"])
    e = d["expect"]
    assert victim == e["victim"] and winner == e["winner"]
    assert rings[victim].tail == e["victim_tail_after"]
    assert rings[winner].head == e["winner_head_after"]
    assert rings[winner].slots[0] == ("a", 1)                 # copies <a|1>
    assert before == e["mask_before"] and "".join(str(mask[i]) for i in range(3)) == e["mask_after"]
    assert rings[victim].hot_rest == e["loser_sees_rest"]
    assert sm.intra_steal({0: rings[0], 2: rings[2]}, mask, loser, d["hot_cutoff"]) is None


def test_fig3_inter_block_steal():
    d = load("fig3_steals.json")["inter"]
    segs = {int(k): sm.ColdSeg(v["top"], v["bottom"]) for k, v in d["victim_block_warps"].items()}
    vw, old_bottom = sm.inter_steal(segs, d["cold_cutoff"])
    e = d["expect"]
    assert vw == e["victim_warp"] and old_bottom == 0
    assert segs[vw].bottom == e["bottom_after"]
    thief = sm.HotRing(128, 0, 0)
    thief.head += e["stolen"]
    assert thief.head == e["thief_head_after"]
    assert segs[vw].cold_rest == e["victim_rest_after"]


def test_kernel_conventions_match_modular_counters():
    """The kernel keeps monotone 16-bit head/tail counters; slot = counter % H and
    hot_rest = (head - tail) mod 2^16 agree with the paper's modular arithmetic."""
    H = 256
    for head in range(0, 70000, 997):
        for rest in (0, 1, 17, 255):
            tail = head - rest
            assert ((head - tail) & 0xFFFF) == rest
            assert (head % H - tail % H) % H == rest % H
