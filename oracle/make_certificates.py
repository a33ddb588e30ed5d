"""Write tests/golden/<cfg>_certificate.json from the O3 subset-DP certificate
(calls only oracle/ and the seeded input generator; TEST INFRASTRUCTURE).

  python -m oracle.make_certificates            # c3, c4, c5 (O3)
  python -m oracle.make_certificates client 14  # O4: the first 14 workflows of c4, per-client levels
  python -m oracle.make_certificates client 16 7  # O4 at the full c4 (n = 16), phase 1 on 7 processes
"""
import dataclasses
import json
import os
import sys
import time

import oracle
from synth import config

GOLD = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests", "golden")


def main():
    for name in ("c3", "c4", "c5"):
        prof, q = config(name)
        c = oracle.dp_certificate(prof, q)
        out = {"config": name, "source": "oracle.dp_certificate (oracle/dpcert.c, O3), seed 0 synth.config",
               "weights": [list(w) for w in q.weights],
               "tseq": c["tseq"].hex(), "eseq": c["eseq"].hex(),
               "best_score64": [b.hex() for b in c["best"]],
               "front_T_E": [[t.hex(), e.hex()] for t, e in c["front"]],
               "front_decimal": [[t, e] for t, e in c["front"]]}
        json.dump(out, open(os.path.join(GOLD, f"{name}_certificate.json"), "w"), indent=1)
        print(name, len(c["front"]), c["best"])


def client(n: int, procs: int = 1):
    """O4 (PER_CLIENT) certificate of the c4 profile's first n workflows with
    c4's G = 8, 4 levels, uncapped clients: the literal per-client reading
    at the largest size O4 can run (n = 14: 5^14 level-vector groups)."""
    prof, q = config("c4")
    q = dataclasses.replace(q, n=n, scope=0, weights=((1, 1), (2, 1), (1, 0), (0, 1)))
    t0 = time.time()
    c = oracle.dp_certificate(prof.subset(n), q, procs=procs)
    wall = time.time() - t0
    out = {"config": f"c4 first {n} workflows, PER_CLIENT", "n": n, "g": q.g, "c": q.c,
           "levels": list(q.levels), "scope": "PER_CLIENT",
           "source": "oracle.dp_certificate (oracle/dpcert.c, O4), seed 0 synth.config('c4').subset(n)",
           "oracle_procs": procs, "oracle_wall_s": round(wall, 1),
           "weights": [list(w) for w in q.weights],
           "tseq": c["tseq"].hex(), "eseq": c["eseq"].hex(),
           "best_score64": [b.hex() for b in c["best"]],
           "front_T_E": [[t.hex(), e.hex()] for t, e in c["front"]],
           "front_decimal": [[t, e] for t, e in c["front"]]}
    json.dump(out, open(os.path.join(GOLD, f"c4_client_n{n}_certificate.json"), "w"), indent=1)
    print(n, len(c["front"]), c["best"])


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[1] == "client":
        client(int(sys.argv[2]), int(sys.argv[3]) if len(sys.argv) > 3 else 1)
    else:
        main()
