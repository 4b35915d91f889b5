"""Writes tests/golden/tiny12_optimum.json by exhaustive enumeration with the CPU oracle only
(oracle/liboracle.so); the GPU exhaustive tiny12 run must reproduce this minimum."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
from oracle import oracle as O  # noqa: E402
from workloads import dag  # noqa: E402

g = dag.tiny12()
best, bx, bo, count = O.bruteforce(g)
out = {"_source": "oracle_bruteforce over 4096 placements x 186 linear extensions of the "
                  "SURVEY.md Appendix B tiny12 fixture (no printed paper value exists)",
       "optimum": best, "schedules": count, "best_x": bx.tolist(), "best_order": bo.tolist()}
json.dump(out, open(os.path.join(os.path.dirname(__file__), "tiny12_optimum.json"), "w"), indent=1)
print(out)
