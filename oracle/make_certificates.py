"""Write tests/golden/<cfg>_certificate.json from the O3 subset-DP certificate
(calls only oracle/ and the seeded input generator; TEST INFRASTRUCTURE).

  python -m oracle.make_certificates
"""
import json
import os

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


if __name__ == "__main__":
    main()
