"""One timed oracle clustering in its own process -- TEST INFRASTRUCTURE ONLY
(bench.py's cpu_baseline / --impl reference legs run several of these at
once to measure the all-core throughput of the oracle as it stands).

  python -m oracle.worker CONFIG DATA_SEED RUN_SEED METRIC

prints one JSON line {"seconds": ..., "iterations": ...}; the data
generation is outside the timed region."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402


def main():
    name, data_seed, run_seed, metric = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
    data, cfg = synth.config_data(name, seed=data_seed)
    data = np.ascontiguousarray(data)
    oracle.lib()
    t = time.perf_counter()
    r = oracle.proclus(data, cfg["k"], cfg["l"], seed=run_seed, metric=metric)
    dt = time.perf_counter() - t
    print(json.dumps({"seconds": dt, "iterations": r.iterations}), flush=True)


if __name__ == "__main__":
    main()
