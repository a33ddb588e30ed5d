import time, json, dataclasses, sys
import oracle
from synth import config
n = int(sys.argv[1]); procs = int(sys.argv[2])
prof, q = config("c4")
q = dataclasses.replace(q, n=n, scope=0, weights=((1, 1), (2, 1), (1, 0), (0, 1)))
t0 = time.time()
if procs > 1:
    off, t, e = oracle.client_fronts_parallel(prof.subset(n), q, procs)
    t1 = time.time(); print("fronts", t1 - t0, "points", t.size, flush=True)
c = oracle.dp_certificate(prof.subset(n), q, procs=procs)
print("total", time.time() - t0, len(c["front"]))
try:
    g = json.load(open(f"tests/golden/c4_client_n{n}_certificate.json"))
    print("golden match", [[a.hex(), b.hex()] for a, b in c["front"]] == g["front_T_E"],
          [b.hex() for b in c["best"]] == g["best_score64"])
except FileNotFoundError:
    pass
