"""Pins for the iteration-warp / range-field model (oracle/iterwarp.py,
PAPER.md §5).  Runs without a GPU."""
import json
import os

from oracle.iterwarp import KEY_MAX, iteration_warp_plan, rf_table


def test_fig6_decisions(golden_dir):
    with open(os.path.join(golden_dir, "fig6.json")) as f:
        g = json.load(f)
    rf = {int(k): v for k, v in g["rf"].items()}
    lof = {int(k): v for k, v in g["leaf_of_max_key"].items()}
    # only the leaves of the RG maxima are given by the figure, and only they decide
    # (the decisions and buffers; this test does not check steps)
    plan = iteration_warp_plan(g["rgs"], lambda k: lof.get(k, 0), rf, g["height"])
    assert [p["mode"] for p in plan] == g["expected"]["modes"]
    assert [p["buffer"] for p in plan] == g["expected"]["buffers"]


def test_rf_table_matches_the_papers_example():
    """height 5, the min key of leaf 6 is 16 -> RF(leaf 1) = 16; with
    3 keys per leaf from leaf 6 on (Fig.6 table: 16, 19, 22, 25, ... 58)."""
    mins = [1, 4, 7, 10, 13] + [16 + 3 * j for j in range(20)]   # leaves 1..25 (positions 0..24)
    rf = rf_table(mins, 5)
    assert rf[0] == 16 and rf[1] == 19 and rf[2] == 22 and rf[3] == 25 and rf[14] == 58
    assert rf[-1] == KEY_MAX


def test_horizontal_steps_and_lazy_repair():
    """Horizontal steps = 1 + links followed; a walk longer than the height
    repairs the start leaf's RF to the min key `height` links right."""
    mins = [10 * i for i in range(40)]             # leaf i holds [10i, 10i + 9]
    leaf_of = lambda k: k // 10                     # noqa: E731
    rf = rf_table(mins, 4)
    # RG1 ends in leaf 2 (RF = min key of leaf 6 = 60); RG2's max 59 <= 60 -> horizontal
    plan = iteration_warp_plan([[5, 21, 29], [30, 45, 59], [200, 210]], leaf_of, rf, 4, mins)
    assert [p["mode"] for p in plan] == ["V", "H", "V"]
    assert plan[0]["steps"] == [4, 4, 4]
    assert plan[1]["steps"] == [2, 3, 4]          # from leaf 2 to leaves 3, 4, 5
    # stale RF (as after splits that inserted leaves): the walk takes > height steps -> repair
    rf2 = list(rf)
    rf2[2] = 1000
    plan = iteration_warp_plan([[25], [95]], leaf_of, rf2, 4, mins)
    assert plan[1]["mode"] == "H" and plan[1]["steps"] == [8]
    assert rf2[2] == mins[6]
