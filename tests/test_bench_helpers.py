"""Host-side helpers of bench.py (no GPU): clock-record parsing and the integer
roofline denominator."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_clocks_summary(tmp_path):
    p = tmp_path / "clk.csv"
    p.write_text(
        "0, 1965, 1965, 700.1, 0x0, Not Active, Not Active, Not Active, Not Active\n"
        "1, 1000, 1965, 300.0, 0x0, Not Active, Not Active, Not Active, Not Active\n"
        "0, 1950, 1965, 720.4, 0x4, Not Active, Not Active, Not Active, Active\n"
        "0, 1965, 1965, 710.0, 0x0, Not Active, Not Active, Not Active, Not Active\n")
    s = bench.clocks_summary(str(p), 0)
    assert s["samples"] == 3 and s["sm_mhz"] == 1965.0 and s["sm_max_mhz"] == 1965.0
    assert s["reasons"] == ["sw_power_cap"]
    assert bench.clocks_summary(str(tmp_path / "missing.csv"), 0)["samples"] == 0


def test_integer_peak_uses_measured_file():
    peak, basis, alu = bench.integer_peak()
    ip = json.load(open(os.path.join(ROOT, "profiles", "int_peaks.json")))
    assert peak == ip["lop3_imad_mixed"] and alu == ip["lop3_alu"]
    assert "measured" in basis
    # the measured mixed rate cannot exceed the issue-slot count at the max clock
    assert peak <= 148 * 4 * 32 * 1965e6 * 1.001


def test_play_match_two_device_players_bookkeeping():
    """play_match with opp_move (the --h2h leg) on two deterministic host movers:
    the lowest-index legal move vs the highest. Colours alternate, so the two
    games are mirror matches; results, disc differences and per-move counts
    must be consistent with a replay under the oracle's rules."""
    import oracle

    def lowest(black, white, to_move, seed):
        own, opp = (black, white) if to_move == 0 else (white, black)
        m = oracle.legal(own, opp)
        return (m & -m).bit_length() - 1, 1

    def highest(black, white, to_move, seed):
        own, opp = (black, white) if to_move == 0 else (white, black)
        return oracle.legal(own, opp).bit_length() - 1, 2

    r = bench.play_match(lowest, 0, 2, 1.0, opp_move=highest)
    assert r["games"] == 2 and sum(r["results"].values()) == 2
    assert r["gpu_playouts_per_move"] == 1 and r["cpu_playouts_per_move"] == 2

    def replay(first_black):  # disc difference of `lowest` in one game
        black, white, to_move = oracle.OPENING_BLACK, oracle.OPENING_WHITE, 0
        while True:
            own, opp = (black, white) if to_move == 0 else (white, black)
            if oracle.legal(own, opp) == 0:
                if oracle.legal(opp, own) == 0:
                    break
                to_move ^= 1
                continue
            lo_turn = (to_move == 0) == first_black
            mv = (lowest if lo_turn else highest)(black, white, to_move, 0)[0]
            f = oracle.flips(own, opp, mv)
            own, opp = own | f | (1 << mv), opp & ~f
            black, white = (own, opp) if to_move == 0 else (opp, own)
            to_move ^= 1
        d = bin(black).count("1") - bin(white).count("1")
        return d if first_black else -d

    want = [replay(True), replay(False)]
    assert r["mean_disc_diff"] == sum(want) / 2
    assert r["results"]["W"] == sum(d > 0 for d in want)
    assert r["point_diff_per_step"][-1] == sum(want) / 2


def test_play_match_depth_per_step():
    """Searchers may return (move, playouts, mean depth); play_match averages the
    depth per game step (ply index) over games, separately for each side
    (Fig. 8 analog). Here side A reports depth = ply index, side B none."""
    import oracle
    seen = []

    def a(black, white, to_move, seed):
        own, opp = (black, white) if to_move == 0 else (white, black)
        m = oracle.legal(own, opp)
        ply = bin(black | white).count("1") - 4  # every move adds one disc
        seen.append(ply)
        return (m & -m).bit_length() - 1, 1, float(ply)

    def b(black, white, to_move, seed):
        own, opp = (black, white) if to_move == 0 else (white, black)
        return oracle.legal(own, opp).bit_length() - 1, 1

    r = bench.play_match(a, 0, 2, 1.0, opp_move=b)
    dp = r["gpu_depth_per_step"]
    assert dp and all(v == float(k) for k, v in dp.items())
    assert sorted(dp) == sorted(set(seen))
    assert r["opp_depth_per_step"] == {}


def test_play_match_seed_base():
    """--sp-seed-base: game g, ply p hands seed_base + 1000 g + p to the
    searcher (the opponent gets +500), so two bases give disjoint seed sets."""
    import oracle
    got = {}

    def mover(tag):
        def f(black, white, to_move, seed):
            got.setdefault(tag, []).append(seed)
            own, opp = (black, white) if to_move == 0 else (white, black)
            m = oracle.legal(own, opp)
            return (m & -m).bit_length() - 1, 1
        return f

    bench.play_match(mover("a"), 0, 2, 1.0, seed_base=100000, opp_move=mover("b"))
    assert min(got["a"]) >= 100000 and max(got["a"]) < 100000 + 2000
    # the opponent's seeds are its plies' bases + 500 (plies alternate sides)
    assert all(100000 <= s - 500 < 100000 + 2000 and (s - 500) % 1000 < 100 for s in got["b"])
    assert set(s - 500 for s in got["b"]).isdisjoint(got["a"])
    seeds_a = sorted(got["a"])
    assert len(set(seeds_a)) == len(seeds_a)
    got.clear()
    bench.play_match(mover("a"), 0, 2, 1.0, opp_move=mover("b"))
    assert max(got["a"]) < 100000


def test_headline_plies_per_s_uses_the_kernel_time():
    """plies_per_s and value divide by the same max-over-ranks device time
    (round 1 divided plies by the shared-tree leg's 500 ms)."""
    h = bench.headline(playouts_total=20 * 4096 * 256, plies_total=20 * 31_433_234, t_ms_max=20 * 0.3795,
                       steps=20)
    assert abs(h["plies_per_s"] - 31_433_234 / 0.3795e-3) < 1e-3 * h["plies_per_s"]
    assert abs(h["value"] - 4096 * 256 / 0.3795e-3) < 1e-3 * h["value"]
    assert h["ms_per_step"] == 0.3795 * 20 / 20
    assert abs(h["plies_per_s"] / h["value"] - 31_433_234 / (4096 * 256)) < 1e-9


def test_roofline_both_fractions():
    r = bench.roofline(plies_per_launch=31_433_234, kern_s=0.3795e-3, peak_ops=3.572317e13, ops_exec=283.8,
                       ops_basis="x", alu_peak=1.85e13, peak_basis="y")
    assert abs(r["frac"] - 31_433_234 * bench.ALG_OPS_PER_PLY / 0.3795e-3 / 3.572317e13) < 1e-9
    assert abs(r["frac_executed"] - 31_433_234 * 283.8 / 0.3795e-3 / 3.572317e13) < 1e-9
    assert r["bound"] == "alu" and r["achieved"] == r["frac"] * r["peak"]


def test_self_launch_cmd():
    assert bench.self_launch_cmd(1, [], {}) is None
    cmd = bench.self_launch_cmd(4, ["--gpus", "4", "--steps", "3"], {})
    assert cmd[1:3] == ["-m", "torch.distributed.run"] and "--nproc-per-node=4" in cmd
    assert "127.0.0.1" in cmd and cmd[-4:] == ["--gpus", "4", "--steps", "3"]
    assert bench.self_launch_cmd(2, [], {"WORLD_SIZE": "2"}) is None
    import pytest
    with pytest.raises(SystemExit):
        bench.self_launch_cmd(2, [], {"WORLD_SIZE": "4"})


def test_kernel_source_hash_is_stable():
    assert bench.kernel_source_hash() == bench.kernel_source_hash() and len(bench.kernel_source_hash()) == 16


def test_play_match_pool_saturation_bookkeeping():
    """Movers may report (refused expansions, slots used, capacity) per search;
    play_match sums the refusals and keeps the fullest pool over the games."""
    import oracle
    calls = []

    def lowest(black, white, to_move, seed):
        own, opp = (black, white) if to_move == 0 else (white, black)
        m = oracle.legal(own, opp)
        calls.append(seed)
        return (m & -m).bit_length() - 1, 1, 2.0, (len(calls) % 3, len(calls), 1000)

    def highest(black, white, to_move, seed):
        own, opp = (black, white) if to_move == 0 else (white, black)
        return oracle.legal(own, opp).bit_length() - 1, 2

    r = bench.play_match(lowest, 0, 2, 1.0, opp_move=highest)
    n = len(calls)
    assert r["gpu_refused_expansions"] == sum(i % 3 for i in range(1, n + 1))
    assert abs(r["gpu_pool_max_fill"] - n / 1000) < 1e-12
    assert r["gpu_depth_per_step"] and all(v == 2.0 for v in r["gpu_depth_per_step"].values())
