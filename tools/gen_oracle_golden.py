"""Write tests/golden/oracle_configs.json: the CPU oracle's results on the five synthetic
configs (test infrastructure; calls only oracle/ and synth/, never the CUDA path).

Per config: the Algorithm 1 partition and its T (k = 1), the exact optimum (C1/C2 full
brute force, C3/C4 the LB-skipping enumeration, same lex order), restart 0 of the
heuristic (T, simulations, walk steps), and for C5 the 65 536-restart winner and its
Slicer sweep.  tests/test_oracle_golden.py checks the oracle still reproduces the file
and that it agrees with the survey's independent scratch values."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import synth  # noqa: E402


def main(out=os.path.join(ROOT, "tests", "golden", "oracle_configs.json")):
    doc = {"source": "tools/gen_oracle_golden.py (oracle/ only; synth/ inputs)", "configs": {}}
    for cfg in synth.ALL_CONFIGS:
        wl = synth.config(cfg)
        M = oracle.Model.from_workload(wl)
        c, v = M.alg1(wl.p)
        e = {"name": wl.name, "n": wl.n, "p": wl.p, "m": wl.m,
             "alg1": {"cuts": [int(x) for x in c], "value": int(v),
                      "T": M.T(wl.p, wl.m, c)}}
        if cfg in (1, 2):
            o = M.exhaustive_parallel(wl.p, wl.m, wl.k_lo, wl.k_hi)
        elif cfg in (3, 4):
            o = M.exhaustive_bnb(wl.p, wl.m, wl.k_lo, wl.k_hi)
        else:
            o = None
        if o is not None:
            e["optimum"] = {"k": [wl.k_lo, wl.k_hi], "T": int(o["T"]), "rank": int(o["rank"]),
                            "k_best": int(o["k"]), "cuts": [int(x) for x in o["cuts"]]}
        h = M.heuristic_restart(wl.p, wl.m, wl.seed or 0x5EED, wl.radius or 2, 0)
        e["heuristic_restart0"] = {"T": int(h["T"]), "sims": int(h["sims"]), "steps": int(h["steps"]),
                                   "cuts": [int(x) for x in h["cuts"]]}
        if cfg == 5:
            hh = M.heuristic_parallel(wl.p, wl.m, wl.seed, wl.radius, 0, wl.restarts)
            T, bk = M.slice_sweep(wl.p, wl.m, hh["cuts"], wl.slice_k_max)
            e["heuristic"] = {"restarts": wl.restarts, "T": int(hh["T"]), "restart": int(hh["restart"]),
                              "cuts": [int(x) for x in hh["cuts"]], "sims": int(hh["sims"]),
                              "slicer_T": [int(x) for x in T], "slicer_best_k": int(bk)}
        doc["configs"][str(cfg)] = e
    with open(out, "w") as fh:
        json.dump(doc, fh, indent=1)
        fh.write("\n")
    print("wrote", out)


if __name__ == "__main__":
    main()
