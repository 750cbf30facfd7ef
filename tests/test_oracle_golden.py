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
