"""Oracle vs hand-worked golden fixtures (tests/golden/README.md)."""
import json
import os

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _name(kind, st, mb, q, k):
    s = "FB"[kind] + f"({st},{mb}"
    if kind == 0 and mb == 0 and k > 1:
        s += f",{q}"
    return s + ")"


def test_handworked_cases(oracle_mod):
    doc = json.load(open(os.path.join(GOLD, "handworked_p2_m2.json")))
    for c in doc["cases"]:
        M = oracle_mod.Model(c["fwd_ns"], c["bwd_ns"], c["act_bytes"], c["link_bytes_per_s"])
        r = M.simulate(c["p"], c["m"], c["cuts"], k=c["k"], want_path=True, want_all=True)
        assert r["T"] == c["T"], c["name"]
        if "master" in c:
            assert r["master"] == c["master"]
        if "path" in c:
            assert [list(o) for o in r["path"]] == c["path"]
        if "ops" in c:
            got = {_name(kind, st, mb, q, c["k"]): [s0, e0] for (st, kind, mb, q, s0, e0) in r["ops"]}
            assert got == c["ops"], c["name"]


def test_table2_encoding():
    doc = json.load(open(os.path.join(GOLD, "table2_gpt2_345m.json")))
    for prt in doc["partitions"]:
        sizes = prt["sublayers"]
        assert sum(sizes) == 50
        for x, l in enumerate(prt["layers"]):
            extra = 1 if x in (0, 3) else 0       # embedding / head sub-layers
            assert sizes[x] == 2 * l + extra
        assert prt["cuts"] == [sum(sizes[:x + 1]) for x in range(3)]
    assert doc["partitions"][0]["cuts"] == [11, 25, 37]
    assert doc["partitions"][1]["cuts"] == [13, 26, 39]


def test_oracle_configs_golden(oracle_mod):
    """tests/golden/oracle_configs.json (written by tools/gen_oracle_golden.py from the
    oracle alone): the oracle still reproduces it -- Algorithm 1, the exact optima of
    C1-C4, every config's restart-0 walk -- and it agrees with the survey's independent
    scratch model (T_dp and optima; the walk counts are checked in
    test_oracle_pins_heuristic.py)."""
    import synth
    doc = json.load(open(os.path.join(GOLD, "oracle_configs.json")))
    for cfg in synth.ALL_CONFIGS:
        g = doc["configs"][str(cfg)]
        wl = synth.config(cfg)
        M = oracle_mod.Model.from_workload(wl)
        c, v = M.alg1(wl.p)
        assert ([int(x) for x in c], v, M.T(wl.p, wl.m, c)) == \
            (g["alg1"]["cuts"], g["alg1"]["value"], g["alg1"]["T"])
        h = M.heuristic_restart(wl.p, wl.m, wl.seed or 0x5EED, wl.radius or 2, 0)
        assert (h["T"], h["sims"], h["steps"], [int(x) for x in h["cuts"]]) == \
            (g["heuristic_restart0"]["T"], g["heuristic_restart0"]["sims"],
             g["heuristic_restart0"]["steps"], g["heuristic_restart0"]["cuts"])
        if "optimum" in g:
            o = (M.exhaustive_parallel(wl.p, wl.m, wl.k_lo, wl.k_hi) if cfg in (1, 2)
                 else M.exhaustive_bnb(wl.p, wl.m, wl.k_lo, wl.k_hi))
            assert (o["T"], o["rank"], o["k"], [int(x) for x in o["cuts"]]) == \
                (g["optimum"]["T"], g["optimum"]["rank"], g["optimum"]["k_best"], g["optimum"]["cuts"])
    # SURVEY.md §8c P15 (independent scratch model) against the committed oracle output
    C = doc["configs"]
    assert C["1"]["optimum"]["T"] == 49664 and C["1"]["optimum"]["rank"] == 60
    assert C["2"]["alg1"]["T"] == 90539622 and C["2"]["alg1"]["cuts"] == [14, 27, 41]
    assert (C["2"]["optimum"]["T"], C["2"]["optimum"]["rank"], C["2"]["optimum"]["k_best"]) == (87232315, 12243, 4)
    assert C["3"]["alg1"]["T"] == 94741098 and C["4"]["alg1"]["T"] == 672610004
    assert C["5"]["alg1"]["T"] == 441984812 and C["5"]["heuristic_restart0"]["T"] == 430480412
    assert C["5"]["heuristic"]["T"] <= C["5"]["heuristic_restart0"]["T"]
