"""Fig. 1 queue microbenchmark sweep
through libatos's atos_queue_bench, i.e. on the worker's own ring code.

Sweeps worker size (thread / warp / CTA), FETCH_SIZE (indices per
leader reservation) and atomicAdd vs CAS reservation over the paper's
three experiments (n threads x 10 pushes / pops / push-then-pop pairs), best of
3 device times, and checks multiset conservation on every push-then-pop run.
One JSON line per point on stdout."""
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_chenbpbyo22_b200 import atos  # noqa: E402


def main():
    rounds = 10
    for lg in (10, 12, 14, 16, 17):
        n = 1 << lg
        for op in ("push", "pop", "push_then_pop"):
            for worker in (1, 32, 512):
                fetches = sorted({f for f in (worker, 128, 32, 8, 1) if f <= worker}, reverse=True)
                for fetch in fetches:
                    for cas in (False, True):
                        if cas and (lg > 14 or fetch != worker):
                            continue          # CAS storms: seconds per launch beyond 2^14 threads
                        best = 1e30
                        ok = True
                        for rep in range(3):
                            check = op == "push_then_pop" and rep == 0
                            ms, popped = atos.queue_bench(worker, op, n, rounds, fetch_size=fetch, reserve_cas=cas,
                                                          popped=check)
                            if check:
                                ok = bool(np.array_equal(np.sort(popped), np.arange(n * rounds, dtype=np.uint32)))
                            best = min(best, ms)
                        ops = n * rounds * (2 if op == "push_then_pop" else 1)
                        print(json.dumps({"op": op, "threads": n, "worker": worker, "fetch": fetch,
                                          "reserve": "cas" if cas else "atomicAdd", "ms": round(best, 5),
                                          "Mops": round(ops / (best * 1e-3) / 1e6, 1),
                                          "conserved": ok if op == "push_then_pop" else None}), flush=True)


if __name__ == "__main__":
    main()
